// k_tbcluster.cuh -- thread-block-cluster backend for conv2d: the hardware
// form of CTA clustering on Blackwell (BASELINE.json north_star "a second
// backend uses Blackwell thread-block clusters with DSMEM and TMA multicast").
//
// A cluster of C vertically adjacent output tiles (cluster dims (1, C, 1)) is
// guaranteed co-scheduled on one GPC.  Each CTA issues ONE TMA load of its 32
// centre rows (40 columns: x0-4 .. x0+35) multicast to every CTA of the
// cluster; rank 0 and rank C-1 also multicast the 8-row boxes above and below
// the cluster.  Every CTA therefore receives the whole cluster region (rows
// r0-8 .. r0+32C+8) into the same shared-memory offsets, and reads its R-row
// halos -- the inter-CTA reuse -- from shared memory that a neighbour's TMA
// filled, instead of re-reading them through L1/L2.  TMA zero-fills
// out-of-range boxes, which gives the image border for free.
// The cluster barrier emits CCTL.IVALL (L1 flush), which is harmless here:
// this backend carries its reuse in shared memory, not L1.
#pragma once
#include <cuda.h>
#include "cc_mem.cuh"
#include "cc_runtime.cuh"
#include "k_stencil.cuh"

namespace cc {

constexpr int TBC_COLS = 40;            // staged columns per row (x0-4 .. x0+35)
constexpr int TBC_ROW_BYTES = TBC_COLS * 4;
constexpr int TBC_HALO = 8;             // halo box height (keeps boxes 128-B aligned)

__device__ __forceinline__ uint32_t cluster_ctarank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// 2D TMA load of box (x, y) multicast to every CTA in `mask` (same smem offset
// and same mbarrier offset in each destination CTA).
__device__ __forceinline__ void tma_load_2d_mc(const CUtensorMap* map, void* dst, uint64_t* bar,
                                               int32_t x, int32_t y, uint16_t mask) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster"
        " [%0], [%1, {%2, %3}], [%4], %5;"
        :: "r"(smem_u32(dst)), "l"(map), "r"(x), "r"(y), "r"(smem_u32(bar)), "h"(mask) : "memory");
}

// Grid (gx, gy_pad) with cluster dims (1, C, 1); dynamic smem =
// tbc_smem_bytes(C): an 8-byte mbarrier, then the region at the next 128-byte
// boundary (TMA destinations must be 128-byte aligned; every box is a multiple
// of 128 bytes, so all box offsets stay aligned).
inline size_t tbc_smem_bytes(int C) { return 256 + (size_t)(2 * TBC_HALO + 32 * C) * TBC_ROW_BYTES; }
template <int R>
__global__ void __launch_bounds__(256) k_conv_tbc(const __grid_constant__ CUtensorMap map_rows,
                                                  const __grid_constant__ CUtensorMap map_halo,
                                                  Sched s, ConvParams<R> p, int32_t C) {
    extern __shared__ __align__(128) uint8_t smem_raw[];
    uint64_t* bar = reinterpret_cast<uint64_t*>(smem_raw);
    const uint32_t sbase = smem_u32(smem_raw);
    float* region = reinterpret_cast<float*>(smem_raw + (((sbase + 16 + 127) & ~127u) - sbase));
    const int rank = (int)cluster_ctarank();
    const int bx = blockIdx.x, by = blockIdx.y;
    const int x0 = bx * 32;
    const int r0 = (by - rank) * 32;           // first output row of the cluster
    const uint16_t mask = (uint16_t)((1u << C) - 1u);
    const uint32_t total = (uint32_t)(2 * TBC_HALO + 32 * C) * TBC_ROW_BYTES;
    if (threadIdx.x == 0) {
        mbar_init(bar, 1);
        fence_mbar_init();
    }
    cluster_sync_all();                         // every barrier initialised before any multicast lands
    if (threadIdx.x == 0) {
        mbar_arrive_tx(bar, total);
        tma_load_2d_mc(&map_rows, region + (TBC_HALO + 32 * rank) * TBC_COLS, bar, x0 - 4, r0 + 32 * rank, mask);
        if (rank == 0) tma_load_2d_mc(&map_halo, region, bar, x0 - 4, r0 - TBC_HALO, mask);
        if (rank == C - 1)
            tma_load_2d_mc(&map_halo, region + (TBC_HALO + 32 * C) * TBC_COLS, bar, x0 - 4, r0 + 32 * C, mask);
    }
    mbar_wait(bar, 0);
    if (by < s.g.gy)
        conv_tile_compute<R>(p, region + (TBC_HALO + 32 * rank - R) * TBC_COLS, bx, by, threadIdx.x);
    if (threadIdx.x == 0 && by < s.g.gy) {
        int32_t lin = by * s.g.gx + bx;
        if (s.census) atomicAdd(s.census + lin, 1u);
        if (s.exec_sm) s.exec_sm[lin] = (int32_t)smid();
    }
    cluster_sync_all();                         // no CTA leaves while cluster traffic may target it
}

}  // namespace cc
