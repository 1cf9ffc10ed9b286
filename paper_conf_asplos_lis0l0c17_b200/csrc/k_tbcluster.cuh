// k_tbcluster.cuh -- thread-block-cluster backend for conv2d: the hardware
// form of CTA clustering on Blackwell (BASELINE.json north_star "a second
// backend uses Blackwell thread-block clusters (__cluster_dims__) with DSMEM
// and TMA").
//
// A cluster of C CTAs (cluster dims (C,1,1)) is co-scheduled by the hardware
// on one GPC -- clustering with no software binding at all.  Clusters are
// persistent: cluster c processes the "units" c, c + NC, c + 2 NC, ... where a
// unit is C vertically adjacent output tiles (bx, C*ub .. C*ub + C-1) and units
// are numbered row-major (ub, bx).  Per unit, CTA k of the cluster
//   1. TMA-loads only its own 32 centre rows (40 columns, x0-4 .. x0+35) into
//      one of two shared-memory buffers (the next unit's load overlaps the
//      current unit's compute); the cluster's outermost CTAs also load the
//      8-row box above / below the cluster;
//   2. tells its neighbours its rows have landed (remote mbarrier arrive),
//      waits for theirs, and copies its R-row halos -- the inter-CTA reuse --
//      straight out of the neighbours' shared memory over DSMEM;
//   3. tells its neighbours it is done reading (remote arrive), so they may
//      refill that buffer two units later, and computes its tile.
// Inside a cluster no halo row is fetched from L2 twice and no cluster-wide
// barrier is needed per unit.  (cluster.sync emits CCTL.IVALL; this backend
// carries its reuse in shared memory, so that is irrelevant anyway.)
#pragma once
#include <cuda.h>
#include "cc_mem.cuh"
#include "cc_runtime.cuh"
#include "k_stencil.cuh"

namespace cc {

constexpr int TBC_COLS = ST_COLS;       // staged columns per row (x0-4 .. x0+35)
constexpr int TBC_ROW_BYTES = TBC_COLS * 4;
#ifndef CC_TBC_HALO
#define CC_TBC_HALO 8
#endif
// halo box height: a multiple of 4 rows (4 x 160 B = 5 x 128 B) keeps every
// TMA destination 128-B aligned; >= R
constexpr int TBC_HALO = CC_TBC_HALO;
static_assert(TBC_HALO % 4 == 0 && TBC_HALO >= 3, "halo box");
constexpr int TBC_ROWS = 2 * TBC_HALO + 32;
constexpr int TBC_BUF_BYTES = TBC_ROWS * TBC_ROW_BYTES;
// output rows per thread: 2 for the HBM-bound 3x3 (4 warps per CTA), 4 for the
// FP32-bound 7x7 (2 warps: each staged row feeds more outputs, as in the agents)
template <int R> constexpr int tbc_rb() { return R >= 3 ? 4 : 2; }
template <int R> constexpr int tbc_threads() { return 256 / tbc_rb<R>(); }
// smem per buffer: [0, 8) top halo box | [8, 40) centre | [40, 48) bottom halo box
inline size_t tbc_smem_bytes(int) { return 256 + 2 * (size_t)TBC_BUF_BYTES; }

__device__ __forceinline__ uint32_t cluster_ctarank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t cluster_id_x() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t nclusters_x() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%nclusterid.x;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// address of the same shared-memory location in CTA `rank` of this cluster
__device__ __forceinline__ uint32_t dsmem_addr(const void* p, uint32_t rank) {
    uint32_t out;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(out) : "r"(smem_u32(p)), "r"(rank));
    return out;
}
__device__ __forceinline__ float4 ld_dsmem4(uint32_t addr) {
    float4 v;
    asm volatile("ld.shared::cluster.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(addr) : "memory");
    return v;
}
// Arrive on the mbarrier at the same offset in CTA `rank`.  Default (CTA-scope)
// semantics on purpose: the data this orders lives in shared memory -- TMA
// writes completed on the producer's own barrier, DSMEM reads are not cached --
// while .release/.acquire.cluster would emit an L1 invalidation (CCTL.IVALL)
// plus a memory barrier on every unit (38 % of stall samples in ncu r03a).
__device__ __forceinline__ void mbar_arrive_remote(uint64_t* bar, uint32_t rank) {
    asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" :: "r"(dsmem_addr(bar, rank)) : "memory");
}
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t parity) { mbar_wait(bar, parity); }

// Persistent grid of NC clusters x C CTAs (1D, cluster dims (C,1,1)),
// tbc_threads<R>() threads, dynamic smem tbc_smem_bytes(C).
template <int R>
__global__ void __launch_bounds__(tbc_threads<R>()) k_conv_tbc(const __grid_constant__ CUtensorMap map_rows,
                                                          const __grid_constant__ CUtensorMap map_halo,
                                                          const __grid_constant__ Sched s,
                                                          const __grid_constant__ ConvParams<R> p, int32_t C) {
    extern __shared__ __align__(128) uint8_t smem_raw[];
    __shared__ uint64_t full[2], ready[2], done[2];
    const uint32_t sbase = smem_u32(smem_raw);
    float* bufs = reinterpret_cast<float*>(smem_raw + (((sbase + 127) & ~127u) - sbase));
    const int rank = (int)cluster_ctarank();
    const int nbrs = (rank > 0 ? 1 : 0) + (rank < C - 1 ? 1 : 0);
    const int gx = s.g.gx, gy = s.g.gy;
    const int ubs = (gy + C - 1) / C;                    // unit rows
    const int units = gx * ubs;
    const int c0 = (int)cluster_id_x(), NC = (int)nclusters_x();
    if (threadIdx.x == 0) {
        for (int b = 0; b < 2; ++b) {
            mbar_init(&full[b], 1);
            if (nbrs) { mbar_init(&ready[b], nbrs); mbar_init(&done[b], nbrs); }
        }
        fence_mbar_init();
    }
    cluster_sync_all();                                  // every barrier of the cluster initialised

    // producer step (thread 0): stage unit `u` of this cluster into buffer b
    auto stage = [&](int u, int b) {
        float* buf = bufs + b * (TBC_BUF_BYTES / 4);
        const int bx = u % gx, ub = u / gx;
        const int x0 = bx * 32, y0 = (ub * C + rank) * 32;
        uint32_t bytes = 32 * TBC_ROW_BYTES;
        if (rank == 0) bytes += TBC_HALO * TBC_ROW_BYTES;
        if (rank == C - 1) bytes += TBC_HALO * TBC_ROW_BYTES;
        mbar_arrive_tx(&full[b], bytes);
        tma_load_2d(buf + TBC_HALO * TBC_COLS, &map_rows, x0 - 4, y0, &full[b]);
        if (rank == 0) tma_load_2d(buf, &map_halo, x0 - 4, y0 - TBC_HALO, &full[b]);
        if (rank == C - 1) tma_load_2d(buf + (TBC_HALO + 32) * TBC_COLS, &map_halo, x0 - 4, y0 + 32, &full[b]);
    };

    int i = 0;
    if (threadIdx.x == 0 && c0 < units) stage(c0, 0);
    for (int u = c0; u < units; u += NC, ++i) {
        const int b = i & 1;
        const uint32_t par = (uint32_t)(i >> 1) & 1u;
        // prefetch the next unit into the other buffer once the neighbours are done with it
        const int un = u + NC;
        if (threadIdx.x == 0 && un < units) {
            if (i >= 1 && nbrs) mbar_wait_cluster(&done[b ^ 1], (uint32_t)((i - 1) >> 1) & 1u);
            stage(un, b ^ 1);
        }
        float* buf = bufs + b * (TBC_BUF_BYTES / 4);
        mbar_wait(&full[b], par);                        // my centre rows (and edge halos) landed
        if (nbrs) {
            if (threadIdx.x == 0) {                      // tell the neighbours
                if (rank > 0) mbar_arrive_remote(&ready[b], rank - 1);
                if (rank < C - 1) mbar_arrive_remote(&ready[b], rank + 1);
            }
            mbar_wait_cluster(&ready[b], par);           // theirs landed too
            for (int idx = threadIdx.x; idx < 2 * R * 10; idx += tbc_threads<R>()) {
                const int side = idx / (R * 10), rem = idx - side * R * 10;
                const int rr = rem / 10, cc = rem - rr * 10;
                if (side == 0 && rank > 0) {             // rows 8-R.. <- rank-1's centre rows 32-R..
                    const float* src = buf + (TBC_HALO + 32 - R + rr) * TBC_COLS + 4 * cc;
                    reinterpret_cast<float4*>(buf + (TBC_HALO - R + rr) * TBC_COLS)[cc] = ld_dsmem4(dsmem_addr(src, rank - 1));
                }
                if (side == 1 && rank < C - 1) {         // rows 40.. <- rank+1's centre rows 0..
                    const float* src = buf + (TBC_HALO + rr) * TBC_COLS + 4 * cc;
                    reinterpret_cast<float4*>(buf + (TBC_HALO + 32 + rr) * TBC_COLS)[cc] = ld_dsmem4(dsmem_addr(src, rank + 1));
                }
            }
            __syncthreads();                             // halos copied (my reads of theirs are done)
            if (threadIdx.x == 0) {
                if (rank > 0) mbar_arrive_remote(&done[b], rank - 1);
                if (rank < C - 1) mbar_arrive_remote(&done[b], rank + 1);
            }
        }
        const int bx = u % gx, by = (u / gx) * C + rank;
        if (by < gy) {
            conv_tile_compute<R, tbc_rb<R>()>(p, buf + (TBC_HALO - R) * TBC_COLS, bx, by, threadIdx.x);
            if (threadIdx.x == 0) {
                const int32_t lin = by * gx + bx;
                if (s.census) atomicAdd(s.census + lin, 1u);
                if (s.exec_sm) s.exec_sm[lin] = (int32_t)smid();
            }
        }
        __syncthreads();                                 // buffer b free for my next use
    }
    cluster_sync_all();                                  // nobody leaves while a neighbour may read it
}

}  // namespace cc
