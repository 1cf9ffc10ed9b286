// k_stencil.cuh -- 5-point Jacobi and 2D cross-correlation tile bodies.
//
// Logical CTA (bx, by) computes the 32 x 32 output tile at rows 32*by..,
// columns 32*bx.. .  The inter-CTA reuse is the halo: the H rows above/below
// and the columns left/right of a tile are the border data of its neighbours
// (the cache-line/algorithm-related classes).
//
// How the tile plus halo (rows y0-H .. y0+31+H, columns x0-4 .. x0+35, i.e.
// 10 aligned 16-byte chunks per row) reaches the consumers (Sched::staging):
//   TMA    one 2D tensor load per tile, L2 -> shared memory, L1 untouched;
//          the image border is zero-filled by the TMA unit (default);
//   L1     cp.async.ca 16-byte chunks: every line also allocates in L1, so a
//          neighbouring tile staged soon after on the same SM finds its halo
//          in L1 -- the paper's inter-CTA L1 reuse, which clustering
//          neighbouring tiles onto one SM (TILE order, Fig. 7) is meant to
//          exploit;
//   direct no staging: consumers load through L1 themselves (plain kernel).
// Consumers: 256 threads; thread (r = ctid/8, c4 = ctid%8) owns the float4 at
// row r, columns 4*c4 .. 4*c4+3 of the tile.
#pragma once
#include "cc_mem.cuh"
#include "cc_runtime.cuh"

namespace cc {

enum : int32_t { STAGE_TMA = 1, STAGE_L1 = 2, STAGE_DIRECT = 3 };
constexpr int ST_COLS = 40;                 // staged floats per row (x0-4 .. x0+35)
// Merged slots: two horizontally adjacent tiles of a cluster in one TMA box
// (x0-4 .. x0+67).  (Runs of four measured 1-5 % slower in round 1: the
// larger slots cost an agent per SM.)
constexpr int ST_MERGE = 2;
constexpr int ST_COLS2 = 32 * ST_MERGE + 8;  // merged slot width in floats (72)

// Split staging for CC_L2_HINT_HALO_LAST: the tile's box as two TMA loads --
// the first 32 rows (evict_first: nothing reads them again after this tile
// and the tile below it) and the last 2H rows (evict_last: the next tile row
// re-reads them as its top halo, about one tile row of the cluster later,
// after the ROW cluster's other traffic has turned L2 over).  t / b: 40-column
// boxes, t2 / b2: the merged 72-column boxes.  Filled by the host only when
// the hint is requested.
struct SplitMaps { CUtensorMap t, b, t2, b2; };

template <int H>
struct HaloTile {
    static constexpr int kRows = 32 + 2 * H;
    static constexpr int kBytes = ((kRows * ST_COLS * 4) + 127) & ~127;
    static constexpr int kBytes2 = ((kRows * ST_COLS2 * 4) + 127) & ~127;   // merged tiles, one box
    // warp-collective: stage the merged box of tiles (bx, by), (bx+1, by) by TMA
    __device__ __forceinline__ static void stage2(int32_t x0, int32_t y0, uint8_t* dst, uint64_t* full, int lane,
                                                  const CUtensorMap* tmap2, int32_t l2_hint,
                                                  const SplitMaps* split = nullptr) {
        stage_commit(full, lane, (uint32_t)(kRows * ST_COLS2 * 4));
        if (lane == 0) {
            if ((l2_hint & L2H_HALO_LAST) && split) {
                tma_load_2d(dst, &split->t2, x0 - 4, y0 - H, full);
                tma_load_2d_h(dst + 32 * ST_COLS2 * 4, &split->b2, x0 - 4, y0 + 32 - H, full, l2_evict_last());
            } else if (l2_hint & L2H_REUSE_LAST) {
                tma_load_2d_h(dst, tmap2, x0 - 4, y0 - H, full, l2_evict_last());
            } else {
                tma_load_2d(dst, tmap2, x0 - 4, y0 - H, full);
            }
        }
    }
    // warp-collective: stage rows y0-H.., columns x0-4.. of `src` (TMA or L1 mode).
    __device__ __forceinline__ static void stage(const float* src, int64_t ld, int32_t rows, int32_t cols,
                                                 int32_t x0, int32_t y0, uint8_t* dst, uint64_t* full, int lane,
                                                 int32_t mode, const CUtensorMap* tmap, int32_t l2_hint = 0,
                                                 const SplitMaps* split = nullptr) {
        if (mode == STAGE_DIRECT) { stage_commit(full, lane, 0); return; }
        if (mode == STAGE_TMA) {
            stage_commit(full, lane, (uint32_t)(kRows * ST_COLS * 4));
            if (lane == 0) {
                // the input is the reused operand (halo rows feed the next tile row)
                if ((l2_hint & L2H_HALO_LAST) && split) {
                    tma_load_2d(dst, &split->t, x0 - 4, y0 - H, full);
                    tma_load_2d_h(dst + 32 * ST_COLS * 4, &split->b, x0 - 4, y0 + 32 - H, full, l2_evict_last());
                } else if (l2_hint & L2H_REUSE_LAST) {
                    tma_load_2d_h(dst, tmap, x0 - 4, y0 - H, full, l2_evict_last());
                } else {
                    tma_load_2d(dst, tmap, x0 - 4, y0 - H, full);
                }
            }
            return;
        }
        const int32_t cols4 = (cols + 3) & ~3;   // last 16-byte chunk stays inside ld
        // lanes 0..29 cover three staged rows (10 chunks each) per step
        const int r0 = lane / 10, cc = lane - r0 * 10;
        const int32_t gx = x0 - 4 + 4 * cc;
        const bool col_ok = lane < 30 && gx >= 0 && gx < cols4;
        if (lane < 30) {
            for (int rr = r0; rr < kRows; rr += 3) {
                const int32_t gy = y0 - H + rr;
                const bool ok = col_ok && gy >= 0 && gy < rows;
                const float* g = ok ? src + (int64_t)gy * ld + gx : src;
                cp_async_ca16(dst + (rr * ST_COLS + 4 * cc) * 4, g, ok ? 16u : 0u);
            }
        }
        cp_async_arrive(full);
        stage_commit(full, lane, 0);
    }
};

__device__ __forceinline__ void store4_masked(float* dst, float4 o, int gx, int cols) {
    if (gx + 4 <= cols) *reinterpret_cast<float4*>(dst) = o;
    else {
        dst[0] = o.x;
        if (gx + 1 < cols) dst[1] = o.y;
        if (gx + 2 < cols) dst[2] = o.z;
    }
}
// the output is the streamed operand: with L2H_STREAM_FIRST its lines leave L2 first
__device__ __forceinline__ void store4_out(float* dst, float4 o, int gx, int cols, int32_t l2_hint) {
    if (!(l2_hint & L2H_STREAM_FIRST)) { store4_masked(dst, o, gx, cols); return; }
    const uint64_t pol = l2_evict_first();
    if (gx + 4 <= cols) st4_h(dst, o, pol);
    else {
        st1_h(dst, o.x, pol);
        if (gx + 1 < cols) st1_h(dst + 1, o.y, pol);
        if (gx + 2 < cols) st1_h(dst + 2, o.z, pol);
    }
}

// ---------------------------------------------------------------------------
// Jacobi 5-point sweep (reading R14, PolyBench jacobi-2d form):
//   b[i][j] = 0.2f * ((((c + w) + e) + s) + n)     on the interior (s = row i+1, n = row i-1),
//   b[i][j] = a[i][j]                               on the boundary.
// fp32, summed in that fixed order with no contraction, so the sweep is
// bit-reproducible against oracle_jacobi5_f32 in every staging mode.
// ---------------------------------------------------------------------------
// Fused peer-memory halo exchange of the slab-sharded sweep (S§8(f)4,
// CC_K_JACOBI5_HALO), in the flag-in-data ("low latency", LL) form: every halo
// value crosses as one 64-bit word {fp32 bits, absolute sweep number}.  The
// thread that computes a slab's first (last) owned row of sweep s also stores
// it, tagged s, into the upper (lower) neighbour's LL buffer of parity s & 1
// -- NVLink peer stores on a multi-GPU box, plain stores for virtual slabs on
// one GPU.  The thread that needs a halo row in sweep s (> 1) polls its own LL
// buffer of parity (s-1) & 1 until every word it needs carries tag s-1.  An
// 8-byte word is written and read in one piece, so the tag vouches for its
// value: no fence on either side (a system-scope fence per tile drains the
// SM's whole store queue and cost more than the exchange saved).  WAR: the
// writer of sweep s+2 first read tag s+1 at the same columns, which the
// neighbour's thread deposited only after (by data dependence) reading the
// sweep-s words being overwritten.  Sweep 1 reads the caller's initial halo
// rows from the slab.  All LL pointers null = the unsharded sweep.
// Only the tile rows next to a halo differ from the plain sweep.  Their
// producer adds one 256-byte bulk copy of the tile's 32 LL words per halo row
// to the stage (same mbarrier as the tile's TMA), so the LL read rides with
// the tile copy instead of stalling anyone; the consumers check the tags in
// shared memory and only re-poll global memory (strong loads) for words
// whose tag is stale.  A word is 8-byte aligned inside a 32-byte sector, so
// no copy can split a value from its tag.  (A consumer-side poll cost ~5 us
// per launch, a producer-side one ~4 us: measured.)
struct JacobiHalo {
    uint64_t* ll;             // mine: [2 parity][2 side][ldl]; side 0 = from up, 1 = from down
    uint64_t* up_ll;          // upper neighbour's LL (I deposit my first owned row into its side 1); null: none
    uint64_t* dn_ll;          // lower neighbour's LL (my last owned row into its side 0); null: none
    int32_t ldl;              // LL row length: cols rounded up to 32 (whole tiles)
    uint32_t sweep;           // absolute sweep number of this launch (1-based)
    int32_t* status;          // optional: 1 = a poll timed out (results invalid)
};
// row0 / row_end: the output row window [row0, row_end) (logical tile row by
// covers rows row0 + 32*by ..); the full sweep has row0 = 0, row_end = rows
struct JacobiParams { CUtensorMap tmap; CUtensorMap tmap2; SplitMaps split; const float* a; float* b; int64_t ld; int32_t rows, cols; int32_t row0, row_end; JacobiHalo h; };

__device__ __forceinline__ uint64_t globaltimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// LL words are accessed at system scope: across GPUs they are NVLink peer
// stores / loads.  (A .gpu-scope build and one without the deposits timed the
// parts of the fused sweep in round 1: identical / -0.5 us.)
#define CC_LL_SCOPE "sys"
__device__ __forceinline__ uint64_t ll_word(float v, uint32_t tag) {
    return ((uint64_t)tag << 32) | (uint64_t)__float_as_uint(v);
}
// deposit 4 consecutive values (16-byte aligned group of 4 words; the first
// `valid` are inside the image) tagged `tag`
__device__ __forceinline__ void ll_store4(uint64_t* dst, float4 o, uint32_t tag, int valid) {
    if (valid >= 4) {
        asm volatile("st.relaxed." CC_LL_SCOPE ".global.v2.u64 [%0], {%1, %2};\n\t"
                     "st.relaxed." CC_LL_SCOPE ".global.v2.u64 [%0+16], {%3, %4};"
                     :: "l"(dst), "l"(ll_word(o.x, tag)), "l"(ll_word(o.y, tag)), "l"(ll_word(o.z, tag)),
                        "l"(ll_word(o.w, tag)) : "memory");
        return;
    }
    const float v[3] = {o.x, o.y, o.z};
    for (int e = 0; e < valid; ++e)
        asm volatile("st.relaxed." CC_LL_SCOPE ".global.u64 [%0], %1;" :: "l"(dst + e), "l"(ll_word(v[e], tag)) : "memory");
}
// poll 4 words until the first `valid` carry `tag`; bounded: after 4 s in
// total (or once *status is set by an earlier timeout) give up and set *status
__device__ __forceinline__ float4 ll_load4(const uint64_t* src, uint32_t tag, int valid, int32_t* status) {
    uint64_t w[4];
    uint64_t t0 = 0;
    for (;;) {
        asm volatile("ld.relaxed." CC_LL_SCOPE ".global.v2.u64 {%0, %1}, [%4];\n\t"
                     "ld.relaxed." CC_LL_SCOPE ".global.v2.u64 {%2, %3}, [%4+16];"
                     : "=l"(w[0]), "=l"(w[1]), "=l"(w[2]), "=l"(w[3]) : "l"(src) : "memory");
        bool ok = true;
#pragma unroll
        for (int e = 0; e < 4; ++e) ok &= e >= valid || (uint32_t)(w[e] >> 32) == tag;
        if (ok) break;
        if (t0 == 0) {
            if (status && *(volatile int32_t*)status) break;      // an earlier poll already gave up
            t0 = globaltimer();
        } else if (globaltimer() - t0 > 4000000000ull) {
            if (status) atomicExch(status, 1);
            break;
        }
        __nanosleep(128);
    }
    return make_float4(__uint_as_float((uint32_t)w[0]), __uint_as_float((uint32_t)w[1]),
                       __uint_as_float((uint32_t)w[2]), __uint_as_float((uint32_t)w[3]));
}
// the 4 words from the stage copy if all carry `tag`, else poll global memory
__device__ __forceinline__ float4 ll_take4(const uint64_t* staged, const uint64_t* src, uint32_t tag, int valid,
                                           int32_t* status) {
    if (staged) {
        const ulonglong2 a = *reinterpret_cast<const ulonglong2*>(staged);
        const ulonglong2 b = *reinterpret_cast<const ulonglong2*>(staged + 2);
        const uint64_t w[4] = {a.x, a.y, b.x, b.y};
        bool ok = true;
#pragma unroll
        for (int e = 0; e < 4; ++e) ok &= e >= valid || (uint32_t)(w[e] >> 32) == tag;
        if (ok)
            return make_float4(__uint_as_float((uint32_t)w[0]), __uint_as_float((uint32_t)w[1]),
                               __uint_as_float((uint32_t)w[2]), __uint_as_float((uint32_t)w[3]));
    }
    return ll_load4(src, tag, valid, status);
}

// PolyBench order: centre, west, east, south (row i+1 = dn), north (row i-1 = up)
__device__ __forceinline__ float4 jacobi_core4(float4 c, float4 up, float4 dn, float lw, float re) {
    float4 o;
    o.x = __fmul_rn(0.2f, __fadd_rn(__fadd_rn(__fadd_rn(__fadd_rn(c.x, lw), c.y), dn.x), up.x));
    o.y = __fmul_rn(0.2f, __fadd_rn(__fadd_rn(__fadd_rn(__fadd_rn(c.y, c.x), c.z), dn.y), up.y));
    o.z = __fmul_rn(0.2f, __fadd_rn(__fadd_rn(__fadd_rn(__fadd_rn(c.z, c.y), c.w), dn.z), up.z));
    o.w = __fmul_rn(0.2f, __fadd_rn(__fadd_rn(__fadd_rn(__fadd_rn(c.w, c.z), re), dn.w), up.w));
    return o;
}
__device__ __forceinline__ float4 jacobi_point4(float4 c, float4 up, float4 dn, float lw, float re,
                                               int gy, int gx, int rows, int cols) {
    float4 o = jacobi_core4(c, up, dn, lw, re);
    const bool row_bd = (gy == 0) || (gy == rows - 1);
    const int cl = cols - 1;
    if (row_bd || gx == 0 || gx == cl) o.x = c.x;
    if (row_bd || gx + 1 == cl) o.y = c.y;
    if (row_bd || gx + 2 == cl) o.z = c.z;
    if (row_bd || gx + 3 == cl) o.w = c.w;
    return o;
}

// HALO = true is the fused peer-halo form (CC_K_JACOBI5_HALO); the plain
// sweep is a separate instantiation, so it carries none of its code.
template <bool HALO>
struct Jacobi5BodyT {
    static constexpr int RB = 2;                  // output rows per consumer thread
    static constexpr int kConsumers = 256 / RB;
    static constexpr int kMerge = HALO ? 1 : ST_MERGE;   // neighbouring tiles per slot (cc_runtime.cuh: MergeOf)
    static constexpr int kTileBytes = HALO ? HaloTile<1>::kBytes : HaloTile<1>::kBytes2;
    static constexpr int kStageBytes = kTileBytes + (HALO ? 2 * 32 * 8 : 0);   // + the two LL halo rows (words)
    static constexpr int kDefaultStages = 4;
    static constexpr int kDefaultBatch = 4;
    static constexpr int kMinAgents = 4;
    static constexpr int kGroups = 2;              // two 4-warp groups consume alternate tiles
    using Params = JacobiParams;
    const JacobiParams& p;   // __grid_constant__ kernel parameter
    int32_t l2h = 0;         // cc_l2_hint bits; set by k_agent only (one-shot kernels keep the literal 0)
    __device__ __forceinline__ explicit Jacobi5BodyT(const JacobiParams& prm) : p(prm) {}

    // fused halo: which halo rows this tile row needs / which owned rows it deposits
    __device__ __forceinline__ bool need_top(int32_t by) const { return HALO && p.h.up_ll && by == 0; }
    __device__ __forceinline__ bool need_bot(int32_t by) const { return HALO && p.h.dn_ll && by == (p.rows - 2) / 32; }
    // Boundary tile rows first: the body visits tile row L = (rows-2)/32 (the
    // lower deposit) right after row 0, then the rest in order -- a fixed
    // bijection on tile rows applied to whatever order the plan gives, so
    // coverage is untouched.  The deposits then land at the start of every
    // sweep, and the next sweep's polls (also at its start) find them: no LL
    // round trip sits in a launch's tail (the classic boundary-first overlap).
    __device__ __forceinline__ int32_t phys_row(int32_t by) const {
        if (!HALO || !p.h.dn_ll) return by;
        const int32_t L = (p.rows - 2) / 32, first = p.h.up_ll ? 1 : 0;
        if (by < first || by > L) return by;
        return by == first ? L : by - 1;
    }

    __device__ __forceinline__ void produce(const Sched& s, int32_t bx, int32_t by, uint8_t* stage, uint64_t* full, int lane) {
        by = phys_row(by);
        if (HALO && p.h.sweep > 1 && s.staging == STAGE_TMA && (need_top(by) || need_bot(by))) {
            // the tile's TMA plus one bulk copy of its 32 LL words per halo row
            const bool top = need_top(by), bot = need_bot(by);
            const int32_t par = (int32_t)((p.h.sweep - 1) & 1u) * 2 * p.h.ldl;
            const uint32_t ll_bytes = (top ? 256u : 0u) + (bot ? 256u : 0u);
            stage_commit(full, lane, (uint32_t)(HaloTile<1>::kRows * ST_COLS * 4) + ll_bytes);
            if (lane == 0) {
                tma_load_2d(stage, &p.tmap, bx * 32 - 4, p.row0 + by * 32 - 1, full);
                uint8_t* extra = stage + kTileBytes;
                if (top) bulk_g2s(extra, p.h.ll + par + bx * 32, 256u, full);
                if (bot) bulk_g2s(extra + 256, p.h.ll + par + p.h.ldl + bx * 32, 256u, full);
            }
            return;
        }
        HaloTile<1>::stage(p.a, p.ld, p.rows, p.cols, bx * 32, p.row0 + by * 32, stage, full, lane, s.staging, &p.tmap,
                           l2h, &p.split);
    }

    // merged slots (plain sweep, TMA staging): tiles (bx, by), (bx+1, by) in one box
    __device__ __forceinline__ bool can_merge(const Sched& s) const { return s.staging == STAGE_TMA; }
    __device__ __forceinline__ void produce_n(const Sched& s, int32_t bx, int32_t by, int n, uint8_t* stage,
                                              uint64_t* full, int lane) {
        if (n >= 2) HaloTile<1>::stage2(bx * 32, p.row0 + by * 32, stage, full, lane, &p.tmap2, l2h, &p.split);
        else produce(s, bx, by, stage, full, lane);
    }
    __device__ __forceinline__ void consume_n(const Sched& s, int32_t bx, int32_t by, int n, const uint8_t* stage,
                                              int ctid) {
        if (n >= 2) {
            consume_at(s, bx, by, stage, ctid, ST_COLS2, 0);
            consume_at(s, bx + 1, by, stage, ctid, ST_COLS2, 32);
        } else {
            consume_at(s, bx, by, stage, ctid, ST_COLS, 0);
        }
    }
    __device__ __forceinline__ void consume(const Sched& s, int32_t bx, int32_t by, const uint8_t* stage, int ctid) {
        consume_at(s, bx, by, stage, ctid, ST_COLS, 0);
    }

    // thread (rows r0 .. r0+RB-1, columns 4*c4 .. 4*c4+3): the RB+2 input rows
    // it touches are read once each.  The staged box has `pitch` floats per row
    // and this tile's columns start `coff` floats in.
    __device__ __forceinline__ void consume_at(const Sched& s, int32_t bx, int32_t by, const uint8_t* stage, int ctid,
                                               int pitch, int coff) {
        by = phys_row(by);
        const int r0 = (ctid >> 3) * RB, c4 = ctid & 7;
        const int gx = bx * 32 + 4 * c4;
        const int gy0 = p.row0 + by * 32 + r0;
        const bool in_col = gx < p.cols;
        float4 row[RB + 2];                        // input rows gy0-1 .. gy0+RB
        float lw[RB], re[RB];
        if (s.staging == STAGE_DIRECT) {
            // plain-kernel form: every load goes through L1 (neighbouring rows are
            // other threads' rows -> L1 hits)
            const float* a = p.a + (int64_t)gy0 * p.ld + gx;
#pragma unroll
            for (int k = 0; k < RB + 2; ++k) {
                const int gy = gy0 - 1 + k;
                row[k] = (in_col && gy >= 0 && gy < p.rows) ? ld_cached4(a + (int64_t)(k - 1) * p.ld) : f4_zero();
            }
#pragma unroll
            for (int j = 0; j < RB; ++j) {
                const int gy = gy0 + j;
                lw[j] = __shfl_up_sync(0xffffffffu, row[j + 1].w, 1, 8);
                re[j] = __shfl_down_sync(0xffffffffu, row[j + 1].x, 1, 8);
                const bool in = in_col && gy < p.rows;
                if (c4 == 0) lw[j] = (in && gx > 0) ? ld_cached(a + (int64_t)j * p.ld - 1) : 0.f;
                if (c4 == 7) re[j] = (in && gx + 4 < p.cols) ? ld_cached(a + (int64_t)j * p.ld + 4) : 0.f;
            }
        } else {
            const float* t = reinterpret_cast<const float*>(stage) + r0 * pitch + coff + 4 + 4 * c4;   // staged row r0 = gy0-1
#pragma unroll
            for (int k = 0; k < RB + 2; ++k) row[k] = *reinterpret_cast<const float4*>(t + k * pitch);
#pragma unroll
            for (int j = 0; j < RB; ++j) {
                lw[j] = t[(j + 1) * pitch - 1];
                re[j] = t[(j + 1) * pitch + 4];
            }
        }
        if (!in_col) return;
        const bool top = need_top(by), bot = need_bot(by);
        if (HALO && (top || bot)) {
            // halo rows of sweep s-1: the LL values (sweep 1: the caller's rows, as staged)
            const uint32_t sw = p.h.sweep;
            const int valid = p.cols - gx < 4 ? p.cols - gx : 4;
            const int32_t par = (int32_t)((sw - 1) & 1u) * 2 * p.h.ldl;
            const uint64_t* extra = reinterpret_cast<const uint64_t*>(stage + kTileBytes);
            if (sw > 1) {
#pragma unroll
                for (int k = 0; k < RB + 2; ++k) {
                    const int gy = gy0 - 1 + k;
                    if (top && gy == 0)
                        row[k] = ll_take4(s.staging == STAGE_TMA ? extra + 4 * c4 : nullptr, p.h.ll + par + gx, sw - 1,
                                          valid, p.h.status);
                    if (bot && gy == p.rows - 1)
                        row[k] = ll_take4(s.staging == STAGE_TMA ? extra + 32 + 4 * c4 : nullptr,
                                          p.h.ll + par + p.h.ldl + gx, sw - 1, valid, p.h.status);
                }
            }
            const int32_t opar = (int32_t)(sw & 1u) * 2 * p.h.ldl;        // parity this sweep deposits into
#pragma unroll
            for (int j = 0; j < RB; ++j) {
                const int gy = gy0 + j;
                if (gy >= p.row_end) break;
                const float4 o = jacobi_point4(row[j + 1], row[j], row[j + 2], lw[j], re[j], gy, gx, p.rows, p.cols);
                store4_masked(p.b + (int64_t)gy * p.ld + gx, o, gx, p.cols);
                if (top && gy == 1) ll_store4(p.h.up_ll + opar + p.h.ldl + gx, o, sw, valid);
                if (bot && gy == p.rows - 2) ll_store4(p.h.dn_ll + opar + gx, o, sw, valid);
            }
            return;
        }
        if (gx >= 1 && gx + 4 <= p.cols - 1 && gy0 >= 1 && gy0 + RB <= p.rows - 1 &&
            gy0 + RB <= p.row_end) {
            // interior block: no boundary cells, plain float4 stores (same arithmetic)
#pragma unroll
            for (int j = 0; j < RB; ++j) {
                float* dst = p.b + (int64_t)(gy0 + j) * p.ld + gx;
                const float4 o = jacobi_core4(row[j + 1], row[j], row[j + 2], lw[j], re[j]);
                if (l2h & L2H_STREAM_FIRST) st4_h(dst, o, l2_evict_first());
                else *reinterpret_cast<float4*>(dst) = o;
            }
            return;
        }
#pragma unroll
        for (int j = 0; j < RB; ++j) {
            const int gy = gy0 + j;
            if (gy >= p.row_end) break;
            store4_out(p.b + (int64_t)gy * p.ld + gx,
                       jacobi_point4(row[j + 1], row[j], row[j + 2], lw[j], re[j], gy, gx, p.rows, p.cols), gx,
                       p.cols, l2h);
        }
    }
    __device__ __forceinline__ void finish(int) {}
};
using Jacobi5Body = Jacobi5BodyT<false>;
using Jacobi5HaloBody = Jacobi5BodyT<true>;

// ---------------------------------------------------------------------------
// K consecutive Jacobi sweeps per launch (reading R32).  The logical CTAs of
// sweeps t+1 .. t+K-1 that need tile (bx, by)'s data are clustered onto the
// agent that holds it, consecutively: the producer stages the tile with a
// K-row / 4-column halo (one TMA box of 40 x (32 + 2K)), the consumer group
// runs sweeps t+1 .. t+K-1 on the shrinking region in shared memory (ping-pong
// between the ring slot it owns and a per-group scratch buffer; redundant
// halo compute, no inter-tile communication) and sweep t+K on the 32 x 32
// tile, which it stores.  HBM sees one read and one write per K sweeps.
// Every point is computed with the single-sweep arithmetic (PolyBench order,
// global boundary copied) from the same inputs, so results are bit-identical
// to K launches of the one-sweep body.
// ---------------------------------------------------------------------------
template <int K>
struct Jacobi5MultiBody {
    static_assert(K >= 2 && K <= 4, "2..4 fused sweeps (the 4-column side halo bounds K)");
    // two output rows per thread (256-thread groups with one row each measured
    // 28 % slower: fewer agents per SM)
    static constexpr int RB = 2;
    static constexpr int kConsumers = 256 / RB;
    static constexpr int kRows = 32 + 2 * K;                    // staged rows
    static constexpr int kMerge = 2;                            // two neighbouring tiles per slot (MergeOf)
    static constexpr int kStageBytes = ((kRows * ST_COLS2 * 4) + 127) & ~127;
    static constexpr int kDirectStageBytes = kStageBytes;     // always TMA-staged
    static constexpr int kDefaultStages = 4;
    static constexpr int kDefaultBatch = 4;
    // three agents per SM: the ring (4 x ~11 KB) and the intermediate-sweep
    // scratch (2 x ~11 KB) fit three per SM anyway, and 3 (not 4) in
    // __launch_bounds__ lets a thread keep 72 registers instead of 56
    static constexpr int kMinAgents = 3;
    static constexpr int kGroups = 2;
    using Params = JacobiParams;
    const JacobiParams& p;
    int32_t l2h = 0;
    __device__ __forceinline__ explicit Jacobi5MultiBody(const JacobiParams& prm) : p(prm) {}

    __device__ __forceinline__ void produce(const Sched&, int32_t bx, int32_t by, uint8_t* stage, uint64_t* full,
                                            int lane) {
        stage_commit(full, lane, (uint32_t)(kRows * ST_COLS * 4));
        if (lane == 0) tma_load_2d(stage, &p.tmap, bx * 32 - 4, by * 32 - K, full);
    }
    // merged slots: tiles (bx, by), (bx+1, by) in one 72-column box
    __device__ __forceinline__ bool can_merge(const Sched&) const { return true; }
    __device__ __forceinline__ void produce_n(const Sched& s, int32_t bx, int32_t by, int n, uint8_t* stage,
                                              uint64_t* full, int lane) {
        if (n < 2) { produce(s, bx, by, stage, full, lane); return; }
        stage_commit(full, lane, (uint32_t)(kRows * ST_COLS2 * 4));
        if (lane == 0) tma_load_2d(stage, &p.tmap2, bx * 32 - 4, by * 32 - K, full);
    }

    // one intermediate sweep S (1 <= S < K) over staged rows [S, kRows - S) and
    // the whole staged width (P / 4 float4 chunks), src -> dst.  Only the
    // region K - S columns / rows inside the box edge is needed; the extra
    // columns are computed from in-bounds neighbours (the adjacent row's ends)
    // and never read by a valid point.  Thread = (chunk, a run of rows): the
    // three rows it needs slide down in registers.  P (the box pitch: one
    // tile or a merged pair) is a template parameter so that the chunk / run
    // split is compile-time; a box with no global-boundary point among those
    // it computes (every box but the image's outer ring) takes the plain
    // 5-point form, without jacobi_point4's per-element boundary selects.
    template <int S, int P>
    __device__ __forceinline__ void sweep(const float* src, float* dst, int32_t bx, int32_t by, int ctid) const {
        constexpr int H = kRows - 2 * S;
        constexpr int nch = P / 4;
        constexpr int runs = kConsumers / nch;                  // row runs that fit the group
        constexpr int rs = (H + runs - 1) / runs;               // rows per run
        constexpr int G = (H + rs - 1) / rs;
        static_assert(rs <= 8, "row run length");
        if (ctid >= G * nch) return;
        const int chunk = ctid % nch, rg = ctid / nch;
        const int r0 = S + rg * rs;
        const int n = r0 + rs <= kRows - S ? rs : kRows - S - r0;
        const int gx0 = bx * 32 - 4, gyb = by * 32 - K;
        const int gx = gx0 + 4 * chunk;
        const float* q = src + 4 * chunk;
        float4 up = *reinterpret_cast<const float4*>(q + (r0 - 1) * P);
        float4 cur = *reinterpret_cast<const float4*>(q + r0 * P);
        const bool interior = gyb + S >= 1 && gyb + kRows - S <= p.rows - 1 && gx0 >= 1 && gx0 + P <= p.cols - 1;
        if (interior) {
#pragma unroll
            for (int k = 0; k < rs; ++k) {
                if (k >= n) break;
                const int r = r0 + k;
                const float4 down = *reinterpret_cast<const float4*>(q + (r + 1) * P);
                const float lw = q[r * P - 1], re = q[r * P + 4];
                *reinterpret_cast<float4*>(dst + r * P + 4 * chunk) = jacobi_core4(cur, up, down, lw, re);
                up = cur;
                cur = down;
            }
        } else {
#pragma unroll
            for (int k = 0; k < rs; ++k) {
                if (k >= n) break;
                const int r = r0 + k;
                const float4 down = *reinterpret_cast<const float4*>(q + (r + 1) * P);
                const float lw = q[r * P - 1], re = q[r * P + 4];
                *reinterpret_cast<float4*>(dst + r * P + 4 * chunk) =
                    jacobi_point4(cur, up, down, lw, re, gyb + r, gx, p.rows, p.cols);
                up = cur;
                cur = down;
            }
        }
    }

    // the last sweep on tile (bx, by) whose columns start coff floats into the box
    __device__ __forceinline__ void final_sweep(const float* F, int pitch, int coff, int32_t bx, int32_t by,
                                                int ctid) const {
        const int r0 = (ctid >> 3) * RB, c4 = ctid & 7;
        const int gx = bx * 32 + 4 * c4, gy0 = by * 32 + r0;
        if (gx >= p.cols) return;
        const float* t = F + (K - 1 + r0) * pitch + coff + 4 + 4 * c4;      // staged row of input row gy0 - 1
        float4 row[RB + 2];
        float lw[RB], re[RB];
#pragma unroll
        for (int k = 0; k < RB + 2; ++k) row[k] = *reinterpret_cast<const float4*>(t + k * pitch);
#pragma unroll
        for (int j = 0; j < RB; ++j) {
            lw[j] = t[(j + 1) * pitch - 1];
            re[j] = t[(j + 1) * pitch + 4];
        }
        const bool inner = gx >= 1 && gx + 4 <= p.cols - 1 && gy0 >= 1 && gy0 + RB <= p.rows - 1;
#pragma unroll
        for (int j = 0; j < RB; ++j) {
            const int gy = gy0 + j;
            if (gy >= p.rows) break;
            float* dst = p.b + (int64_t)gy * p.ld + gx;
            if (inner) *reinterpret_cast<float4*>(dst) = jacobi_core4(row[j + 1], row[j], row[j + 2], lw[j], re[j]);
            else store4_masked(dst, jacobi_point4(row[j + 1], row[j], row[j + 2], lw[j], re[j], gy, gx, p.rows,
                                                  p.cols), gx, p.cols);
        }
    }

    // sweeps 1 .. K-1 on the box, ping-ponging X -> Y -> X ...
    template <int P>
    __device__ __forceinline__ void sweeps(float* X, float* Y, int32_t bx, int32_t by, int ctid) const {
        sweep<1, P>(X, Y, bx, by, ctid);
        consumer_sync<kConsumers>();
        if constexpr (K >= 3) { sweep<2, P>(Y, X, bx, by, ctid); consumer_sync<kConsumers>(); }
        if constexpr (K >= 4) { sweep<3, P>(X, Y, bx, by, ctid); consumer_sync<kConsumers>(); }
    }

    __device__ __forceinline__ void consume_n(const Sched&, int32_t bx, int32_t by, int n, const uint8_t* stage,
                                              int ctid) {
        __shared__ __align__(16) float s_scr[kGroups][kRows * ST_COLS2];   // float4 reads in sweep K
        float* X = reinterpret_cast<float*>(const_cast<uint8_t*>(stage));   // the group owns its slot
        float* Y = s_scr[(threadIdx.x - PRODUCER_THREADS) / kConsumers];
        const float* F = (K & 1) ? X : Y;                          // holds sweep K-1
        if (n >= 2) {
            sweeps<ST_COLS2>(X, Y, bx, by, ctid);
            final_sweep(F, ST_COLS2, 0, bx, by, ctid);
            final_sweep(F, ST_COLS2, 32, bx + 1, by, ctid);
        } else {
            sweeps<ST_COLS>(X, Y, bx, by, ctid);
            final_sweep(F, ST_COLS, 0, bx, by, ctid);
        }
        // K even: sweep K read the scratch buffer, which the group's next task
        // overwrites in its first sweep -- every thread must be done with it
        if constexpr (!(K & 1)) consumer_sync<kConsumers>();
    }
    __device__ __forceinline__ void consume(const Sched& s, int32_t bx, int32_t by, const uint8_t* stage, int ctid) {
        consume_n(s, bx, by, 1, stage, ctid);
    }
    __device__ __forceinline__ void finish(int) {}
};

// ---------------------------------------------------------------------------
// 2D cross-correlation with a (2R+1)^2 filter (reading R15):
//   out[i][j] = sum_{a,b} w[a+R][b+R] * in[i+a][j+b]   interior, else 0.
// The filter lives in the kernel parameter bank (constant-bank operands).
// ---------------------------------------------------------------------------
template <int R>
struct ConvParams { CUtensorMap tmap; CUtensorMap tmap2; SplitMaps split; const float* in; float* out; int64_t ld; int32_t rows, cols; float w[(2 * R + 1) * (2 * R + 1)]; };

// Thread ctid computes RB vertically adjacent rows x 4 columns of the tile
// (256/RB threads per tile).  Each staged input row is read once (3 LDS.128)
// and feeds every output row it is a tap of: RB = 2 cuts the shared-memory
// reads per output by 33 % (3x3) / 43 % (7x7) -- the conv is otherwise
// shared-memory-bandwidth bound.  The summation order per output is the
// filter's row-major tap order, as in the oracle.
// Staged rows as one contiguous box: row rr (input row y0 - R + rr) at base + rr * pitch.
struct ContigRows {
    const float* base;
    int pitch;
    __device__ __forceinline__ const float* operator()(int rr) const { return base + rr * pitch; }
};

// The tile's arithmetic, into registers: thread ctid's RB x 4 outputs.
template <int R, int RB, class RowPtr>
__device__ __forceinline__ void conv_tile_acc(const ConvParams<R>& p, const RowPtr& rowp, int ctid,
                                              float (&acc)[RB][4]) {
    // rowp(rr) points at the staged row holding input row y0 - R + rr, column x0 - 4
    constexpr int K = 2 * R + 1;
    const int r0 = (ctid >> 3) * RB, c4 = ctid & 7;
#pragma unroll
    for (int j = 0; j < RB; ++j)
#pragma unroll
        for (int e = 0; e < 4; ++e) acc[j][e] = 0.f;
#pragma unroll
    for (int ir = 0; ir < K + RB - 1; ++ir) {           // staged rows r0 .. r0+K+RB-2
        const float4* row = reinterpret_cast<const float4*>(rowp(r0 + ir) + 4 * c4);
        float4 q0 = row[0], q1 = row[1], q2 = row[2];
        const float win[12] = {q0.x, q0.y, q0.z, q0.w, q1.x, q1.y, q1.z, q1.w, q2.x, q2.y, q2.z, q2.w};
#pragma unroll
        for (int j = 0; j < RB; ++j) {
            const int dy = ir - j;                        // tap row of output row r0+j
            if (dy < 0 || dy >= K) continue;
#pragma unroll
            for (int dx = 0; dx < K; ++dx) {
                const float wt = p.w[dy * K + dx];
#pragma unroll
                for (int e = 0; e < 4; ++e) acc[j][e] = fmaf(wt, win[4 + e + dx - R], acc[j][e]);
            }
        }
    }
}

// ... and out to global memory (interior outputs only; the border stays 0)
template <int R, int RB>
__device__ __forceinline__ void conv_tile_store(const ConvParams<R>& p, int32_t bx, int32_t by, int ctid,
                                                const float (&acc)[RB][4], int32_t l2_hint = 0) {
    const int r0 = (ctid >> 3) * RB, c4 = ctid & 7;
    const int gx = bx * 32 + 4 * c4;
    if (gx >= p.cols) return;
    {
        // interior thread block of outputs (every output of its RB x 4 block
        // has a full window): plain float4 stores, no per-element masks
        const int gy0 = by * 32 + r0;
        if (gx >= R && gx + 4 <= p.cols - R && gy0 >= R && gy0 + RB <= p.rows - R) {
#pragma unroll
            for (int j = 0; j < RB; ++j) {
                float* dst = p.out + (int64_t)(gy0 + j) * p.ld + gx;
                const float4 o = make_float4(acc[j][0], acc[j][1], acc[j][2], acc[j][3]);
                if (l2_hint & L2H_STREAM_FIRST) st4_h(dst, o, l2_evict_first());
                else *reinterpret_cast<float4*>(dst) = o;
            }
            return;
        }
    }
#pragma unroll
    for (int j = 0; j < RB; ++j) {
        const int gy = by * 32 + r0 + j;
        if (gy >= p.rows) break;
        const bool row_in = gy >= R && gy < p.rows - R;
        float4 o;
        o.x = (row_in && gx + 0 >= R && gx + 0 < p.cols - R) ? acc[j][0] : 0.f;
        o.y = (row_in && gx + 1 >= R && gx + 1 < p.cols - R) ? acc[j][1] : 0.f;
        o.z = (row_in && gx + 2 >= R && gx + 2 < p.cols - R) ? acc[j][2] : 0.f;
        o.w = (row_in && gx + 3 >= R && gx + 3 < p.cols - R) ? acc[j][3] : 0.f;
        store4_out(p.out + (int64_t)gy * p.ld + gx, o, gx, p.cols, l2_hint);
    }
}

template <int R, int RB = 1, class RowPtr>
__device__ __forceinline__ void conv_tile_compute_rows(const ConvParams<R>& p, const RowPtr& rowp,
                                                       int32_t bx, int32_t by, int ctid, int32_t l2_hint = 0) {
    float acc[RB][4];
    conv_tile_acc<R, RB>(p, rowp, ctid, acc);
    conv_tile_store<R, RB>(p, bx, by, ctid, acc, l2_hint);
}

template <int R, int RB = 1>
__device__ __forceinline__ void conv_tile_compute(const ConvParams<R>& p, const float* rows_base,
                                                  int32_t bx, int32_t by, int ctid, int32_t l2_hint = 0,
                                                  int pitch = ST_COLS) {
    conv_tile_compute_rows<R, RB>(p, ContigRows{rows_base, pitch}, bx, by, ctid, l2_hint);
}

template <int R>
struct Conv2dBody {
    // output rows per consumer thread: the 7x7 filter is FP32-issue bound, so
    // each thread takes 4 rows (784 FFMA per task against a fixed per-task
    // overhead of ~150 instructions per warp); the 3x3 is HBM bound
    // (8 rows per thread -- twice the FFMA per shared-memory load -- with 2 or
    // 4 one-warp groups measured 20-35 % slower in round 2, gpurun_out r10g)
    static constexpr int RB = R >= 3 ? 4 : 2;
    static constexpr int kConsumers = 256 / RB;
    // two neighbouring tiles per slot for the HBM-bound 3x3 (cc_runtime.cuh:
    // MergeOf); the FP32-bound 7x7 gains nothing from the shared halo and
    // measured 12 % slower merged
    static constexpr int kMerge = R >= 3 ? 1 : ST_MERGE;
    static constexpr int kStageBytes = kMerge > 1 ? HaloTile<R>::kBytes2 : HaloTile<R>::kBytes;
    static constexpr int kDirectStageBytes = HaloTile<R>::kBytes;  // the direct path stages into its own slot
    // Two consumer groups per agent (alternate tiles).  One scheduler warp per
    // two groups: with four 2-warp groups per agent (7x7) the single producer,
    // which gets only its fair share of issue slots, could not keep them fed
    // (measured 0.91x -> 0.99x of default order with two groups).
    static constexpr int kGroups = 2;
    static constexpr int kDefaultStages = 2 * kGroups; // two slots per group: the next tile lands while one computes
    static constexpr int kDefaultBatch = 4;
    // agents per SM: 3x3 4 (56 registers, no spill; measured 5 % faster than
    // 5 with spills), 7x7 6 (56 registers)
    static constexpr int kMinAgents = R >= 3 ? 6 : 4;
    using Params = ConvParams<R>;
    const ConvParams<R>& p;  // __grid_constant__ kernel parameter (filter in the param bank)
    int32_t l2h = 0;         // cc_l2_hint bits; set by k_agent only (one-shot kernels keep the literal 0)
    __device__ __forceinline__ explicit Conv2dBody(const ConvParams<R>& prm) : p(prm) {}

    __device__ __forceinline__ void produce(const Sched& s, int32_t bx, int32_t by, uint8_t* stage, uint64_t* full, int lane) {
        HaloTile<R>::stage(p.in, p.ld, p.rows, p.cols, bx * 32, by * 32, stage, full, lane, s.staging, &p.tmap, l2h,
                           &p.split);
    }
    // plain-kernel form of the staging: the consumers stage the tile themselves
    // through L1, into this task's ring slot (the group owns it until it
    // releases it)
    __device__ __forceinline__ void direct_stage(int32_t bx, int32_t by, const uint8_t* stage, int ctid) {
        auto& s_in = *reinterpret_cast<float4 (*)[HaloTile<R>::kRows][ST_COLS / 4]>(const_cast<uint8_t*>(stage));
        const int x0 = bx * 32, y0 = by * 32;
        for (int idx = ctid; idx < HaloTile<R>::kRows * 10; idx += kConsumers) {
            const int rr = idx / 10, cc = idx - rr * 10;
            const int gy = y0 - R + rr, gx = x0 - 4 + 4 * cc;
            float4 v = f4_zero();
            if (gy >= 0 && gy < p.rows && gx >= 0 && gx < p.cols) v = ld_cached4(p.in + (int64_t)gy * p.ld + gx);
            s_in[rr][cc] = v;
        }
        consumer_sync<kConsumers>();
        // (no trailing barrier: the slot is reused only after every warp of the
        // group has released it)
    }
    __device__ __forceinline__ void consume(const Sched& s, int32_t bx, int32_t by, const uint8_t* stage, int ctid) {
        if (s.staging == STAGE_DIRECT) {
            direct_stage(bx, by, stage, ctid);
            if constexpr (R < 3) {             // 3x3: a second copy of the tile code for the direct path
                conv_tile_compute<R, RB>(p, reinterpret_cast<const float*>(stage), bx, by, ctid, l2h);
                return;
            }
        }
        // 7x7: one instance of the tile code for both staging paths (the direct
        // path staged into this same slot).  Two unrolled copies are 2 x 784
        // FFMA of instruction footprint; the single copy makes every 7x7 agent
        // 3.5 % faster (agent ROW 0.1635 -> 0.1577 ms, same box A/B,
        // profiles/r07/diag/suite_convbody_*).  The 3x3 keeps two copies (its
        // identity order measured 1.8 % slower with one).
        conv_tile_compute<R, RB>(p, reinterpret_cast<const float*>(stage), bx, by, ctid, l2h);
    }
    // merged slots (TMA staging): tiles (bx, by), (bx+1, by) from one box
    __device__ __forceinline__ bool can_merge(const Sched& s) const { return s.staging == STAGE_TMA; }
    __device__ __forceinline__ void produce_n(const Sched& s, int32_t bx, int32_t by, int n, uint8_t* stage,
                                              uint64_t* full, int lane) {
        if (n >= 2) HaloTile<R>::stage2(bx * 32, by * 32, stage, full, lane, &p.tmap2, l2h, &p.split);
        else produce(s, bx, by, stage, full, lane);
    }
    __device__ __forceinline__ void consume_n(const Sched& s, int32_t bx, int32_t by, int n, const uint8_t* stage,
                                              int ctid) {
        if (n >= 2) {
            // one instance of the tile code, run n times (two unrolled copies would
            // not fit the register budget of the resident agents)
            const float* b = reinterpret_cast<const float*>(stage);
#pragma unroll 1
            for (int k = 0; k < n; ++k) conv_tile_compute<R, RB>(p, b + 32 * k, bx + k, by, ctid, l2h, ST_COLS2);
        } else {
            consume(s, bx, by, stage, ctid);
        }
    }
    __device__ __forceinline__ void finish(int) {}
};

}  // namespace cc
