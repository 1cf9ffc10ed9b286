// k_tbcluster.cuh -- thread-block-cluster backend for conv2d: the hardware
// form of CTA clustering on Blackwell (BASELINE.json north_star: "a second
// backend uses Blackwell thread-block clusters (__cluster_dims__) with DSMEM
// and TMA multicast").
//
// A cluster of C CTAs (cluster dims (C,1,1)) is co-scheduled by the hardware
// on one GPC -- clustering with no software binding at all.  Clusters are
// persistent: cluster c processes the units c, c + NC, c + 2 NC, ... where a
// unit is C vertically adjacent output tile rows of TW horizontally adjacent
// 32 x 32 tiles (CTA k of the cluster computes tile row C*ub + k).
//
// The inter-CTA reuse -- the 2R input rows straddling the boundary between
// vertically adjacent tiles, which both tiles read -- is fetched from L2
// ONCE per cluster and delivered to both CTAs by one TMA multicast
// (cp.async.bulk.tensor ... .multicast::cluster, ctaMask = the two CTAs).
// Each CTA's stage holds three regions:
//     X[0], X[1]   2R-row boundary boxes
//     C            its 32 - 2R interior rows (a plain TMA load, itself only)
// The boundary between CTA b and b+1 lands in region X[b & 1] of BOTH CTAs
// (a multicast writes the same shared-memory offset in every destination),
// which is CTA b's bottom and CTA b+1's top boundary; CTA k therefore reads
// its top boundary from X[(k-1) & 1] and its bottom one from X[k & 1], and the
// tile code maps each staged row to its region (ParityRows).  The cluster's
// outermost boundaries are loaded by CTA 0 / CTA C-1 for themselves.
//
// Pipeline (per CTA, 2 consumer groups alternating units, 2 stages each,
// warp-specialised like the agents):
//   warp 0 lane 0 (producer)  for stage s of unit i: wait empty[s] (this CTA
//     and CTA k+1 -- the other receiver of its multicast -- released the
//     stage), arm full[s] with the bytes this CTA receives, issue its
//     interior load and its bottom-boundary multicast (CTA 0 also its top);
//   consumer group            wait full[s], compute its tiles into registers,
//     release the stage -- a local arrive on empty[s] and a remote arrive on
//     CTA k-1's empty[s] (mbarrier.arrive.release.cluster; the producer of a
//     CTA with a lower neighbour waits with .acquire.cluster): the WAR order
//     between this CTA's shared-memory reads and its neighbour's next
//     multicast into them -- then store the outputs.
// No CTA reads another's shared memory: all data arrives by TMA and is
// observed through the CTA's own full barrier (complete_tx), the standard
// async-proxy pattern.  A multicast may complete_tx on a peer's full[s]
// before the peer armed it (the transaction count goes transiently
// negative); it cannot target an earlier phase, since the issuer waited for
// the peer's release of that stage, which follows the peer's consumption of
// the stage's previous phase.
#pragma once
#include <cuda.h>
#include "cc_mem.cuh"
#include "cc_runtime.cuh"
#include "k_stencil.cuh"

namespace cc {

#ifndef CC_TBC_SPG
#define CC_TBC_SPG 2                          // stages per consumer group (round-2 A/B)
#endif
#ifndef CC_TBC_TW3
#define CC_TBC_TW3 2                          // 3x3 tiles per CTA per unit (round-2 A/B)
#endif
constexpr int TBC_GROUPS = 2;                 // consumer groups, alternate units
constexpr int TBC_STAGES = CC_TBC_SPG * TBC_GROUPS;

template <int R, int TW>
struct TbcGeom {
    static constexpr int kCols = 32 * TW + 8;                     // staged floats per row (x0-4 ..)
    static constexpr int kRowB = kCols * 4;
    static constexpr int kB = 2 * R;                              // boundary box rows
    static constexpr int kC = 32 - 2 * R;                         // interior rows
    static constexpr int kRegB = ((kB * kRowB) + 127) & ~127;     // 128-byte aligned regions
    static constexpr int kCenB = ((kC * kRowB) + 127) & ~127;
    static constexpr int kStageB = 2 * kRegB + kCenB;             // X[0] | X[1] | C
    static constexpr uint32_t kRecvBytes = (uint32_t)((32 + 2 * R) * kRowB);   // per CTA per stage
    static constexpr int kRB = R >= 3 ? 4 : 2;                    // output rows per consumer thread
    static constexpr int kConsumers = 256 / kRB;                  // per group (one tile's threads)
    static constexpr int kThreads = TBC_GROUPS * kConsumers + 32;
};
template <int R> constexpr int tbc_tw() { return R >= 3 ? 1 : CC_TBC_TW3; }   // 3x3: two tiles per CTA per unit
template <int R> constexpr int tbc_threads() { return TbcGeom<R, tbc_tw<R>()>::kThreads; }
template <int R> inline size_t tbc_smem_bytes() { return 128 + (size_t)TBC_STAGES * TbcGeom<R, tbc_tw<R>()>::kStageB; }

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
// Stage release to the producer of CTA `rank`, and the producer's wait.
// Default: cluster-scope release / acquire (the PTX memory model's guarantee
// for ordering this CTA's shared-memory reads before the peer's next async
// write into them).  CC_TBC_CTA_SCOPE=1 (diagnostic build) uses the plain
// forms CUTLASS's multicast pipelines use (mbarrier.arrive.shared::cluster,
// default semantics) to measure what the cluster-scope fences cost.
#ifndef CC_TBC_CTA_SCOPE
#define CC_TBC_CTA_SCOPE 0
#endif
__device__ __forceinline__ void mbar_arrive_remote_release(uint64_t* bar, uint32_t rank) {
    if constexpr (CC_TBC_CTA_SCOPE)
        asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" :: "r"(dsmem_addr(bar, rank)) : "memory");
    else
        asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" :: "r"(dsmem_addr(bar, rank))
                     : "memory");
}
__device__ __forceinline__ void mbar_arrive_release_cluster(uint64_t* bar) {
    if constexpr (CC_TBC_CTA_SCOPE)
        mbar_arrive(bar);
    else
        asm volatile("mbarrier.arrive.release.cluster.shared::cta.b64 _, [%0];" :: "r"(smem_u32(bar)) : "memory");
}
// wait with cluster-scope acquire: the remote releases above happen-before what follows
__device__ __forceinline__ void mbar_wait_acquire_cluster(uint64_t* bar, uint32_t parity) {
    if constexpr (CC_TBC_CTA_SCOPE) {
        mbar_wait(bar, parity);
        return;
    }
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAITC_%=:\n\t"
        "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1, %2;\n\t"
        "@!p bra WAITC_%=;\n}" :: "r"(smem_u32(bar)), "r"(parity), "r"(1000000u) : "memory");
}
// 2D TMA load of box (x, y) multicast to the CTAs in `mask`, each at this
// CTA's `dst` offset, completion counted on the barrier at `bar`'s offset in each
__device__ __forceinline__ void tma_load_2d_mc(void* dst, const void* tmap, int32_t x, int32_t y, uint64_t* bar,
                                               uint16_t mask) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.multicast::cluster"
                 " [%0], [%1, {%2, %3}], [%4], %5;"
                 :: "r"(smem_u32(dst)), "l"(tmap), "r"(x), "r"(y), "r"(smem_u32(bar)), "h"(mask) : "memory");
}

// staged row rr (input row y0 - R + rr) of CTA k: top boundary rows [0, 2R)
// in X[(k-1)&1], interior rows [2R, 32) in C, bottom boundary rows [32, 32+2R) in X[k&1]
struct ParityRows {
    const float* top;
    const float* cen;
    const float* bot;
    int pitch, b, c;      // b = 2R, c = 32
    __device__ __forceinline__ const float* operator()(int rr) const {
        return rr < b ? top + rr * pitch : rr < c ? cen + (rr - b) * pitch : bot + (rr - c) * pitch;
    }
};

// Persistent grid of NC clusters x C CTAs (1D, cluster dims (C,1,1)),
// tbc_threads<R>() threads, dynamic smem tbc_smem_bytes<R>().
// map_c: box (kCols x (32 - 2R)), map_b: box (kCols x 2R).
template <int R>
__global__ void __launch_bounds__(tbc_threads<R>()) k_conv_tbc(const __grid_constant__ CUtensorMap map_c,
                                                          const __grid_constant__ CUtensorMap map_b,
                                                          const __grid_constant__ Sched s,
                                                          const __grid_constant__ ConvParams<R> p, int32_t C) {
    constexpr int TW = tbc_tw<R>();
    using G = TbcGeom<R, TW>;
    extern __shared__ uint8_t smem_raw[];
    __shared__ uint64_t full[TBC_STAGES], empty[TBC_STAGES];
    uint8_t* ring = ring_base(smem_raw);
    const int k = (int)cluster_ctarank();
    const int gx = s.g.gx, gy = s.g.gy;
    const int ucols = (gx + TW - 1) / TW;                // unit columns
    const int ubs = (gy + C - 1) / C;                    // unit rows
    const int units = ucols * ubs;
    const int c0 = (int)cluster_id_x(), NC = (int)nclusters_x();
    const bool has_next = k < C - 1;
    if (threadIdx.x == 0) {
        for (int b = 0; b < TBC_STAGES; ++b) {
            mbar_init(&full[b], 1);
            mbar_init(&empty[b], has_next ? 2 : 1);      // the owning group + CTA k+1's
        }
        fence_mbar_init();
    }
    cluster_sync_all();                                  // every barrier of the cluster initialised

    if (threadIdx.x < 32) {
        // ---- producer
        if (threadIdx.x == 0) {
            const uint16_t mask = (uint16_t)((1u << k) | (has_next ? 1u << (k + 1) : 0u));
            int i = 0;
            for (int u = c0; u < units; u += NC, ++i) {
                const int st = i % TBC_STAGES;
                if (i >= TBC_STAGES) {
                    const uint32_t ph = (uint32_t)((i / TBC_STAGES) - 1) & 1u;
                    if (has_next) mbar_wait_acquire_cluster(&empty[st], ph);     // a peer releases too
                    else mbar_wait(&empty[st], ph);
                }
                uint8_t* stage = ring + (size_t)st * G::kStageB;
                const int x0 = (u % ucols) * 32 * TW, y0 = ((u / ucols) * C + k) * 32;
                mbar_arrive_tx(&full[st], G::kRecvBytes);
                tma_load_2d(stage + 2 * G::kRegB, &map_c, x0 - 4, y0 + R, &full[st]);     // interior
                if (k == 0)                                                                  // cluster top
                    tma_load_2d(stage + G::kRegB, &map_b, x0 - 4, y0 - R, &full[st]);      // X[1]
                // bottom boundary into X[k & 1]: shared with CTA k+1 (its top) by one
                // multicast; a cluster's last CTA loads its own
                if (has_next) tma_load_2d_mc(stage + (k & 1) * G::kRegB, &map_b, x0 - 4, y0 + 32 - R, &full[st], mask);
                else tma_load_2d(stage + (k & 1) * G::kRegB, &map_b, x0 - 4, y0 + 32 - R, &full[st]);
            }
        }
    } else {
        // ---- consumers: group grp takes units i = grp, grp + G, ...
        const int grp = (threadIdx.x - 32) / G::kConsumers;
        const int ctid = (threadIdx.x - 32) % G::kConsumers;
        int i = grp;
        for (int u = c0 + grp * NC; u < units; u += TBC_GROUPS * NC, i += TBC_GROUPS) {
            const int st = i % TBC_STAGES;
            mbar_wait(&full[st], (uint32_t)(i / TBC_STAGES) & 1u);
            const uint8_t* stage = ring + (size_t)st * G::kStageB;
            const float* top = reinterpret_cast<const float*>(stage + ((k - 1) & 1) * G::kRegB);
            const float* bot = reinterpret_cast<const float*>(stage + (k & 1) * G::kRegB);
            const float* cen = reinterpret_cast<const float*>(stage + 2 * G::kRegB);
            const int bx0 = (u % ucols) * TW, by = (u / ucols) * C + k;
            // all TW tiles into registers, release the stage, then store: the
            // release's cluster-scope fence then has no fresh stores to drain
            float acc[TW][G::kRB][4];
#pragma unroll
            for (int t = 0; t < TW; ++t) {
                const ParityRows rows{top + 32 * t, cen + 32 * t, bot + 32 * t, G::kCols, 2 * R, 32};
                conv_tile_acc<R, G::kRB>(p, rows, ctid, acc[t]);
            }
            consumer_sync<G::kConsumers>();              // every thread of the group is done reading
            if (ctid == 0) {
                mbar_arrive(&empty[st]);
                if (k > 0) mbar_arrive_remote_release(&empty[st], (uint32_t)(k - 1));
            }
            if (by < gy) {
#pragma unroll
                for (int t = 0; t < TW; ++t) {
                    const int bx = bx0 + t;
                    if (bx >= gx) break;
                    conv_tile_store<R, G::kRB>(p, bx, by, ctid, acc[t]);
                    if (ctid == 0) {
                        const int32_t lin = by * gx + bx;
                        if (s.census) atomicAdd(s.census + lin, 1u);
                        if (s.exec_sm) s.exec_sm[lin] = (int32_t)smid();
                    }
                }
            }
        }
    }
    cluster_sync_all();                                  // no CTA leaves while a peer may still signal it
}

}  // namespace cc
