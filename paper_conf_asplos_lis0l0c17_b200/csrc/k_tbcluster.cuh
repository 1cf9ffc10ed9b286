// k_tbcluster.cuh -- thread-block-cluster backend for conv2d: the hardware
// form of CTA clustering on Blackwell (BASELINE.json north_star "a second
// backend uses Blackwell thread-block clusters (__cluster_dims__) with DSMEM
// and TMA").
//
// A cluster of C vertically adjacent output tiles (cluster dims (1, C, 1)) is
// co-scheduled by the hardware on one GPC -- clustering without any software
// binding.  Each CTA loads only its own 32 centre rows (one 2D TMA load, 40
// columns x0-4 .. x0+35) into shared memory; after a cluster barrier it pulls
// its R-row halos -- the inter-CTA reuse -- straight out of its neighbours'
// shared memory over DSMEM (ld.shared::cluster), so inside a cluster no halo
// row is fetched from L2 twice.  Only the cluster's outermost CTAs load a halo
// box from global memory (TMA, zero-filled at the image border).
// The cluster barrier emits CCTL.IVALL (L1 flush), which is harmless here:
// this backend carries its reuse in shared memory, not L1.
#pragma once
#include <cuda.h>
#include "cc_mem.cuh"
#include "cc_runtime.cuh"
#include "k_stencil.cuh"

namespace cc {

constexpr int TBC_COLS = ST_COLS;       // staged columns per row (x0-4 .. x0+35)
constexpr int TBC_ROW_BYTES = TBC_COLS * 4;
constexpr int TBC_HALO = 8;             // halo box height (keeps every TMA box 128-B aligned)
constexpr int TBC_ROWS = 2 * TBC_HALO + 32;
// smem: [0, 8) top halo box | [8, 40) centre | [40, 48) bottom halo box
inline size_t tbc_smem_bytes(int) { return 256 + (size_t)TBC_ROWS * TBC_ROW_BYTES; }

__device__ __forceinline__ uint32_t cluster_ctarank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
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

// Grid (gx, gy_pad) with cluster dims (1, C, 1); 256 threads; dynamic smem
// tbc_smem_bytes(C).
template <int R>
__global__ void __launch_bounds__(256) k_conv_tbc(const __grid_constant__ CUtensorMap map_rows,
                                                  const __grid_constant__ CUtensorMap map_halo,
                                                  const __grid_constant__ Sched s,
                                                  const __grid_constant__ ConvParams<R> p, int32_t C) {
    extern __shared__ __align__(128) uint8_t smem_raw[];
    uint64_t* bar = reinterpret_cast<uint64_t*>(smem_raw);
    const uint32_t sbase = smem_u32(smem_raw);
    float* region = reinterpret_cast<float*>(smem_raw + (((sbase + 16 + 127) & ~127u) - sbase));
    const int rank = (int)cluster_ctarank();
    const int bx = blockIdx.x, by = blockIdx.y;
    const int x0 = bx * 32, y0 = by * 32;
    if (threadIdx.x == 0) {
        mbar_init(bar, 1);
        fence_mbar_init();
        uint32_t bytes = 32 * TBC_ROW_BYTES;
        if (rank == 0) bytes += TBC_HALO * TBC_ROW_BYTES;
        if (rank == C - 1) bytes += TBC_HALO * TBC_ROW_BYTES;
        mbar_arrive_tx(bar, bytes);
        tma_load_2d(region + TBC_HALO * TBC_COLS, &map_rows, x0 - 4, y0, bar);
        if (rank == 0) tma_load_2d(region, &map_halo, x0 - 4, y0 - TBC_HALO, bar);
        if (rank == C - 1) tma_load_2d(region + (TBC_HALO + 32) * TBC_COLS, &map_halo, x0 - 4, y0 + 32, bar);
    }
    __syncthreads();
    mbar_wait(bar, 0);
    cluster_sync_all();                          // every centre tile of the cluster has landed
    // halo rows from the neighbours' centre rows (DSMEM), R rows x 10 float4 each side
    for (int idx = threadIdx.x; idx < 2 * R * 10; idx += 256) {
        const int side = idx / (R * 10), rem = idx - side * R * 10;
        const int rr = rem / 10, cc = rem - rr * 10;
        if (side == 0 && rank > 0) {             // my rows 8-R.. <- rank-1's centre rows 32-R..
            const float* src = region + (TBC_HALO + 32 - R + rr) * TBC_COLS + 4 * cc;
            reinterpret_cast<float4*>(region + (TBC_HALO - R + rr) * TBC_COLS)[cc] = ld_dsmem4(dsmem_addr(src, rank - 1));
        }
        if (side == 1 && rank < C - 1) {         // my rows 40.. <- rank+1's centre rows 0..
            const float* src = region + (TBC_HALO + rr) * TBC_COLS + 4 * cc;
            reinterpret_cast<float4*>(region + (TBC_HALO + 32 + rr) * TBC_COLS)[cc] = ld_dsmem4(dsmem_addr(src, rank + 1));
        }
    }
    cluster_sync_all();                          // halos copied: neighbours may now leave/overwrite
    if (by < s.g.gy)
        conv_tile_compute<R>(p, region + (TBC_HALO - R) * TBC_COLS, bx, by, threadIdx.x);
    if (threadIdx.x == 0 && by < s.g.gy) {
        const int32_t lin = by * s.g.gx + bx;
        if (s.census) atomicAdd(s.census + lin, 1u);
        if (s.exec_sm) s.exec_sm[lin] = (int32_t)smid();
    }
}

}  // namespace cc
