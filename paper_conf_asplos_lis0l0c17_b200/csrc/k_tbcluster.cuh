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
// ONCE and delivered to both CTAs of a pair (CTAs 2j and 2j+1 of the
// cluster) by one TMA multicast (cp.async.bulk.tensor ... .multicast::cluster,
// ctaMask = the pair).  A multicast writes the same shared-memory offset in
// every destination, so the pair uses mirrored layouts around the shared box:
//
//   even CTA (upper tile)   [ own box: 32 rows | B: Hb rows ]
//   odd CTA  (lower tile)                      [ B: Hb rows | own box: 32 rows ]
//
// B (Hb = 2R rounded up to 4 rows, keeping every TMA destination 128-byte
// aligned) sits at the same offset in both; the odd CTA's ring is the even
// one's shifted by 32 rows, so consecutive stages tile the buffer with one
// stride (32 + Hb rows) in both.  Each CTA's staged rows are contiguous, so
// the tile code is the agents' (ContigRows), and each CTA issues one 32-row
// box per unit (the even one also the Hb-row multicast).  A cluster's
// outermost boundaries, and those between pairs, are loaded by each CTA for
// itself.
//
// Pipeline (per CTA, 2 consumer groups alternating units, 2 stages each,
// warp-specialised like the agents):
//   warp 0 lane 0 (producer)  for stage s of unit i: wait empty[s] (this CTA
//     released it and, for an even CTA, so did its partner -- the other
//     receiver of its multicast), arm full[s] with the bytes this CTA
//     receives, issue its own 32-row box (and, even CTAs, the B multicast);
//   consumer group            wait full[s], compute its tiles into registers,
//     release the stage -- a local arrive on empty[s] and, odd CTAs, a
//     remote arrive on the partner's empty[s] (mbarrier.arrive.release.cluster;
//     the even producer waits with .acquire.cluster): the WAR order between
//     the odd CTA's shared-memory reads of B and the partner's next
//     multicast into it -- then store the outputs.
// No CTA reads another's shared memory: all data arrives by TMA and is
// observed through the CTA's own full barrier (complete_tx), the standard
// async-proxy pattern.  A multicast may complete_tx on the partner's full[s]
// before the partner armed it (the transaction count goes transiently
// negative); it cannot target an earlier phase, since the issuer waited for
// the partner's release of that stage, which follows the partner's
// consumption of the stage's previous phase.
#pragma once
#include <cuda.h>
#include "cc_mem.cuh"
#include "cc_runtime.cuh"
#include "k_stencil.cuh"

namespace cc {

// Two consumer groups alternate units, two stages each, and a 3x3 unit is two
// tiles wide: the measured best (round 2: 3 or 4 stages per group, fewer CTAs
// per SM, 12-28 % slower; one-tile units 30 % slower; profiles/r10/exp/tbc_*).
constexpr int TBC_GROUPS = 2;
constexpr int TBC_STAGES = 2 * TBC_GROUPS;

template <int R, int TW>
struct TbcGeom {
    static constexpr int kCols = 32 * TW + 8;                     // staged floats per row (x0-4 ..)
    static constexpr int kRowB = kCols * 4;
    static constexpr int kHb = (2 * R + 3) & ~3;                  // shared box rows (>= 2R, multiple of 4)
    static constexpr int kLead = kHb / 2 - R;                     // unused rows before a CTA's first staged row
    static constexpr int kStageRows = 32 + kHb;
    static constexpr int kStageB = kStageRows * kRowB;            // stride of the ring (both parities)
    static constexpr uint32_t kRecvBytes = (uint32_t)((32 + kHb) * kRowB);    // per CTA per stage
    static constexpr int kRB = R >= 3 ? 4 : 2;                    // output rows per consumer thread
    static constexpr int kConsumers = 256 / kRB;                  // per group (one tile's threads)
    static constexpr int kThreads = TBC_GROUPS * kConsumers + 32;
    static_assert(kStageB % 128 == 0 && (32 * kRowB) % 128 == 0 && (kHb * kRowB) % 128 == 0, "TMA alignment");
};
template <int R> constexpr int tbc_tw() { return R >= 3 ? 1 : 2; }   // 3x3: two tiles per CTA per unit
template <int R> constexpr int tbc_threads() { return TbcGeom<R, tbc_tw<R>()>::kThreads; }
template <int R> inline size_t tbc_smem_bytes() {
    using G = TbcGeom<R, tbc_tw<R>()>;
    return 128 + (size_t)TBC_STAGES * G::kStageB + (size_t)32 * G::kRowB;   // + the odd CTAs' 32-row shift
}

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
// Stage release to the producer of CTA `rank`, and the producer's wait:
// cluster-scope release / acquire, the PTX memory model's guarantee for
// ordering this CTA's shared-memory reads before the peer's next async write
// into them.  (The plain CTA-scope forms were measured slower as well as
// weaker, and are not built.)
__device__ __forceinline__ void mbar_arrive_remote_release(uint64_t* bar, uint32_t rank) {
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" :: "r"(dsmem_addr(bar, rank))
                 : "memory");
}
__device__ __forceinline__ void mbar_arrive_release_cluster(uint64_t* bar) {
    asm volatile("mbarrier.arrive.release.cluster.shared::cta.b64 _, [%0];" :: "r"(smem_u32(bar)) : "memory");
}
// wait with cluster-scope acquire: the remote releases above happen-before what follows
__device__ __forceinline__ void mbar_wait_acquire_cluster(uint64_t* bar, uint32_t parity) {
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

// Persistent grid of NC clusters x C CTAs (1D, cluster dims (C,1,1)),
// tbc_threads<R>() threads, dynamic smem tbc_smem_bytes<R>().
// map_c: box (kCols x 32), map_b: box (kCols x Hb), map_f: box (kCols x (32 + Hb)).
template <int R>
__global__ void __launch_bounds__(tbc_threads<R>()) k_conv_tbc(const __grid_constant__ CUtensorMap map_c,
                                                          const __grid_constant__ CUtensorMap map_b,
                                                          const __grid_constant__ CUtensorMap map_f,
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
    const bool odd = k & 1;
    const bool partner = !odd && k + 1 < C;              // even CTA with a lower partner: it multicasts B
    uint8_t* base = ring + (odd ? (size_t)32 * G::kRowB : 0);
    if (threadIdx.x == 0) {
        for (int b = 0; b < TBC_STAGES; ++b) {
            mbar_init(&full[b], 1);
            mbar_init(&empty[b], partner ? 2 : 1);       // the owning group (+ the partner's)
        }
        fence_mbar_init();
    }
    cluster_sync_all();                                  // every barrier of the cluster initialised

    if (threadIdx.x < 32) {
        // ---- producer
        if (threadIdx.x == 0) {
            const uint16_t mask = (uint16_t)((1u << k) | (partner ? 1u << (k + 1) : 0u));
            int i = 0;
            for (int u = c0; u < units; u += NC, ++i) {
                const int st = i % TBC_STAGES;
                if (i >= TBC_STAGES) {
                    const uint32_t ph = (uint32_t)((i / TBC_STAGES) - 1) & 1u;
                    if (partner) mbar_wait_acquire_cluster(&empty[st], ph);      // the partner releases too
                    else mbar_wait(&empty[st], ph);
                }
                uint8_t* stage = base + (size_t)st * G::kStageB;
                const int x0 = (u % ucols) * 32 * TW, y0 = ((u / ucols) * C + k) * 32;
                mbar_arrive_tx(&full[st], G::kRecvBytes);
                if (!odd) {
                    // own rows [y0 - Hb/2, y0 + 32 - Hb/2), then B = the Hb rows
                    // centred on the boundary below (multicast to the partner)
                    const int yb = y0 + 32 - G::kHb / 2;
                    if (partner) {
                        tma_load_2d(stage, &map_c, x0 - 4, yb - 32, &full[st]);
                        tma_load_2d_mc(stage + 32 * G::kRowB, &map_b, x0 - 4, yb, &full[st], mask);
                    } else {                                 // no partner: own rows and B as one box
                        tma_load_2d(stage, &map_f, x0 - 4, yb - 32, &full[st]);
                    }
                } else {
                    // B arrives from the partner; own rows [y0 + Hb/2, y0 + Hb/2 + 32)
                    tma_load_2d(stage + G::kHb * G::kRowB, &map_c, x0 - 4, y0 + G::kHb / 2, &full[st]);
                }
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
            // staged row rr = input row y0 - R + rr, contiguous from here in both parities
            const float* rows0 = reinterpret_cast<const float*>(base + (size_t)st * G::kStageB) + G::kLead * G::kCols;
            const int bx0 = (u % ucols) * TW, by = (u / ucols) * C + k;
            // all TW tiles into registers, release the stage, then store: the
            // release's cluster-scope fence then has no fresh stores to drain
            float acc[TW][G::kRB][4];
#pragma unroll
            for (int t = 0; t < TW; ++t) conv_tile_acc<R, G::kRB>(p, ContigRows{rows0 + 32 * t, G::kCols}, ctid, acc[t]);
            consumer_sync<G::kConsumers>();              // every thread of the group is done reading
            if (ctid == 0) {
                mbar_arrive(&empty[st]);
                if (odd) mbar_arrive_remote_release(&empty[st], (uint32_t)(k - 1));
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
