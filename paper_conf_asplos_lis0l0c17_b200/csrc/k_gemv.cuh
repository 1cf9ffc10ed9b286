// k_gemv.cuh -- tile body shared by the tiled matvec and ATAX / BICG / MVT.
//
// Logical CTA (bx, by) owns the TR x TC tile A[TR*by .., TC*bx ..] of a
// row-major fp32 matrix (Listing 2 layout: bx indexes the input
// vector B[idx], by the output C[idy]).  It contributes
//   ROW product:  out_r[rows of by] += A_tile   . vc[cols of bx]   (A x)
//   COL product:  out_c[cols of bx] += A_tile^T . vr[rows of by]   (A^T y)
// This is the cache-line-related class of Table 2 (ATX/MVT/BC).
//
// Data movement:
//   * the A tile (streamed, no reuse) is staged by the producer warp with ONE
//     2D TMA load straight into shared memory (UTMALDG; it never touches L1,
//     the B200 form of the paper's bypass §4.3(II); ragged edges zero-filled);
//   * the vc / vr slices -- the inter-CTA shared data -- are read by the
//     consumers with L1-allocating loads, so tasks of one SM that share bx (vc)
//     or by (vr) hit L1;
//   * partial out_r (out_c) sums are carried in registers across consecutive
//     tasks of one agent with the same by (bx) and flushed to L2 with one
//     (vector) RED only when the row (column) changes -- temporal inter-CTA
//     reuse kept on chip.  Under the default backend every CTA is a fresh task,
//     so it flushes every time: same code, no clustering.
//
// Consumer mapping (256 threads = 8 warps): a tile row is covered by LPR =
// min(32, TC/4) lanes, each holding FPL = TC/(4 LPR) float4 columns; a warp
// covers RPW = 32/LPR rows per pass and runs NP = TR/(8 RPW) passes.  Row sums
// reduce inside a warp (shuffles only); column sums only need the other warps
// at a column flush, which clustering makes rare.
#pragma once
#include "cc_mem.cuh"
#include "cc_runtime.cuh"

namespace cc {

struct GemvParams {
    CUtensorMap tmap;  // A as an n x m fp32 tensor, box TC x TR (filled by the launcher)
    const float* A; int64_t lda; int32_t m, n;
    const float* vc;   // ROW-product input, n entries
    const float* vr;   // COL-product input, m entries
    float* out_r;      // m entries, accumulated
    float* out_c;      // n entries, accumulated
};

template <int TR, int TC, bool DO_ROW, bool DO_COL>
struct GemvBody {
    static constexpr int kConsumers = 256;
    static constexpr int kStageBytes = TR * TC * 4;
    static constexpr int kDefaultStages = 2;
    static constexpr int kDefaultBatch = TC >= 256 ? 2 : 1;
    static constexpr int kMinAgents = 3;
    static constexpr int kGroups = 1;
    static constexpr int CW = TC / 4;                    // float4 columns per row
    static constexpr int LPR = CW < 32 ? CW : 32;        // lanes per row
    static constexpr int FPL = CW / LPR;                 // float4 per lane per row
    static constexpr int RPW = 32 / LPR;                 // rows per warp pass
    static constexpr int NP = TR / (8 * RPW);            // passes
    static_assert(TC % 4 == 0 && CW % LPR == 0 && 32 % LPR == 0 && TR % (8 * RPW) == 0 && NP >= 1, "tile shape");
    using Params = GemvParams;

    const GemvParams& p;   // the __grid_constant__ kernel parameter (TMA needs its address)
    int32_t l2h = 0;         // cc_l2_hint bits; set by k_agent only (one-shot kernels keep the literal 0)
    int32_t cur_ti, cur_tj;
    float racc[NP];
    float4 cacc[FPL];

    __device__ __forceinline__ explicit GemvBody(const GemvParams& prm) : p(prm), cur_ti(-1), cur_tj(-1) {
#pragma unroll
        for (int k = 0; k < NP; ++k) racc[k] = 0.f;
#pragma unroll
        for (int f = 0; f < FPL; ++f) cacc[f] = f4_zero();
    }
    // tile-local row of (warp, pass, sub-row) and float4 column of (lane, f)
    __device__ __forceinline__ static int trow(int warp, int k, int sub) { return (k * RPW + sub) * 8 + warp; }
    __device__ __forceinline__ static int tcol4(int cl, int f) { return f * LPR + cl; }

    // ---- producer: one 2D TMA load of the whole tile (OOB rows/cols zero-filled)
    __device__ __forceinline__ void produce(const Sched& s, int32_t bx, int32_t by, uint8_t* stage, uint64_t* full, int lane) {
        if (s.staging == 3) { stage_commit(full, lane, 0); return; }   // direct: consumers load A
        stage_commit(full, lane, (uint32_t)kStageBytes);
        if (lane == 0) {
            if (l2h & L2H_STREAM_FIRST) tma_load_2d_h(stage, &p.tmap, bx * TC, by * TR, full, l2_evict_first());
            else tma_load_2d(stage, &p.tmap, bx * TC, by * TR, full);
        }
    }

    // ---- ROW flush: warp-level sum over the LPR lanes of each row, one RED per row
    __device__ __forceinline__ void flush_row(int ctid) {
        const int warp = ctid >> 5, lane = ctid & 31, sub = lane / LPR, cl = lane % LPR;
#pragma unroll
        for (int k = 0; k < NP; ++k) {
            float v = racc[k];
#pragma unroll
            for (int o = LPR / 2; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o, LPR);
            const int row = cur_ti * TR + trow(warp, k, sub);
            if (cl == 0 && row < p.m) red_add(p.out_r + row, v);
            racc[k] = 0.f;
        }
    }

    // ---- COL flush: sum cacc over the 8 * RPW row slots, one vector RED per 4 columns
    __device__ __forceinline__ void flush_col(int ctid) {
        __shared__ float4 s_col[DO_COL ? 8 * RPW : 1][DO_COL ? CW : 1];
        const int warp = ctid >> 5, lane = ctid & 31, sub = lane / LPR, cl = lane % LPR;
#pragma unroll
        for (int f = 0; f < FPL; ++f) s_col[warp * RPW + sub][tcol4(cl, f)] = cacc[f];
        consumer_sync<kConsumers>();
        for (int c4 = ctid; c4 < CW; c4 += kConsumers) {
            float4 v = s_col[0][c4];
#pragma unroll
            for (int g = 1; g < 8 * RPW; ++g) {
                const float4 u = s_col[g][c4];
                v.x += u.x; v.y += u.y; v.z += u.z; v.w += u.w;
            }
            const int col = cur_tj * TC + c4 * 4;
            if (col < p.n) {
                if (col + 4 <= p.n) red_add4(p.out_c + col, v);
                else {
                    red_add(p.out_c + col, v.x);
                    if (col + 1 < p.n) red_add(p.out_c + col + 1, v.y);
                    if (col + 2 < p.n) red_add(p.out_c + col + 2, v.z);
                }
            }
        }
        consumer_sync<kConsumers>();
#pragma unroll
        for (int f = 0; f < FPL; ++f) cacc[f] = f4_zero();
    }

    // ---- consumers: one logical CTA from the staged tile
    __device__ __forceinline__ void consume(const Sched& s, int32_t bx, int32_t by, const uint8_t* stage, int ctid) {
        if (DO_ROW && by != cur_ti) { if (cur_ti >= 0) flush_row(ctid); cur_ti = by; }
        if (DO_COL && bx != cur_tj) { if (cur_tj >= 0) flush_col(ctid); cur_tj = bx; }
        const int warp = ctid >> 5, lane = ctid & 31, sub = lane / LPR, cl = lane % LPR;
        const int col0 = bx * TC, row0 = by * TR;
        const bool direct = s.staging == 3;
        const bool hf = l2h & L2H_STREAM_FIRST, hl = l2h & L2H_REUSE_LAST;
        auto vec4 = [&](const float* q) { return hl ? ld_cached4_h(q, l2_evict_last()) : ld_cached4(q); };
        auto vec1 = [&](const float* q) { return hl ? ld_cached_h(q, l2_evict_last()) : ld_cached(q); };
        auto a4 = [&](const float* q) { return hf ? ld_stream4_h(q, l2_evict_first()) : ld_stream4(q); };
        if (col0 + TC <= p.n && row0 + TR <= p.m) {
            // interior tile: no bounds anywhere in the hot loop
            float4 xv[FPL];
            float rv[NP];
#pragma unroll
            for (int f = 0; f < FPL; ++f) xv[f] = DO_ROW ? vec4(p.vc + col0 + tcol4(cl, f) * 4) : f4_zero();
#pragma unroll
            for (int k = 0; k < NP; ++k) rv[k] = DO_COL ? vec1(p.vr + row0 + trow(warp, k, sub)) : 0.f;
            if (direct) {
                // plain-kernel form: issue every A load of the tile first (NP*FPL
                // independent 16-byte loads in flight per thread), then reduce
                float4 av[NP][FPL];
                const float* base = p.A + (int64_t)row0 * p.lda + col0;
                if constexpr (NP * FPL == 8) {
                    float4 v8[8];
                    const float* ptr[8];
#pragma unroll
                    for (int q = 0; q < 8; ++q)
                        ptr[q] = base + (int64_t)trow(warp, q / FPL, sub) * p.lda + tcol4(cl, q % FPL) * 4;
                    if (hf) ld_stream4_x8_h(v8, ptr, l2_evict_first());
                    else ld_stream4_x8(v8, ptr);
#pragma unroll
                    for (int q = 0; q < 8; ++q) av[q / FPL][q % FPL] = v8[q];
                } else if constexpr ((NP * FPL) % 4 == 0) {
                    if (hf) {
#pragma unroll
                        for (int q = 0; q < NP * FPL; ++q)
                            av[q / FPL][q % FPL] = ld_stream4_h(base + (int64_t)trow(warp, q / FPL, sub) * p.lda +
                                                                tcol4(cl, q % FPL) * 4, l2_evict_first());
                    } else
#pragma unroll
                    for (int q = 0; q < NP * FPL; q += 4) {
                        const int k0 = q / FPL, f0 = q % FPL, k1 = (q + 1) / FPL, f1 = (q + 1) % FPL;
                        const int k2 = (q + 2) / FPL, f2 = (q + 2) % FPL, k3 = (q + 3) / FPL, f3 = (q + 3) % FPL;
                        ld_stream4_x4(av[k0][f0], av[k1][f1], av[k2][f2], av[k3][f3],
                                      base + (int64_t)trow(warp, k0, sub) * p.lda + tcol4(cl, f0) * 4,
                                      base + (int64_t)trow(warp, k1, sub) * p.lda + tcol4(cl, f1) * 4,
                                      base + (int64_t)trow(warp, k2, sub) * p.lda + tcol4(cl, f2) * 4,
                                      base + (int64_t)trow(warp, k3, sub) * p.lda + tcol4(cl, f3) * 4);
                    }
                } else {
#pragma unroll
                    for (int k = 0; k < NP; ++k)
#pragma unroll
                        for (int f = 0; f < FPL; ++f)
                            av[k][f] = hf ? ld_stream4_h(base + (int64_t)trow(warp, k, sub) * p.lda + tcol4(cl, f) * 4,
                                                         l2_evict_first())
                                          : ld_stream4_batched(base + (int64_t)trow(warp, k, sub) * p.lda + tcol4(cl, f) * 4);
                }
#pragma unroll
                for (int k = 0; k < NP; ++k)
#pragma unroll
                    for (int f = 0; f < FPL; ++f) accumulate(k, f, av[k][f], xv[f], rv[k]);
                return;
            }
#pragma unroll
            for (int k = 0; k < NP; ++k)
#pragma unroll
                for (int f = 0; f < FPL; ++f)
                    accumulate(k, f, reinterpret_cast<const float4*>(stage)[trow(warp, k, sub) * CW + tcol4(cl, f)],
                               xv[f], rv[k]);
            return;
        }
        // ragged edge tile.  Staged tiles are zero-filled past m / n by the TMA
        // unit; only the vector reads (and direct loads) need bounds.
        float4 xv[FPL];
#pragma unroll
        for (int f = 0; f < FPL; ++f) {
            const int col = col0 + tcol4(cl, f) * 4;
            xv[f] = f4_zero();
            if (DO_ROW && col < p.n) {
                if (col + 4 <= p.n) xv[f] = vec4(p.vc + col);
                else {
                    xv[f].x = vec1(p.vc + col);
                    if (col + 1 < p.n) xv[f].y = vec1(p.vc + col + 1);
                    if (col + 2 < p.n) xv[f].z = vec1(p.vc + col + 2);
                }
            }
        }
#pragma unroll
        for (int k = 0; k < NP; ++k) {
            const int r = trow(warp, k, sub);
            if (row0 + r >= p.m) continue;
            const float rv = DO_COL ? vec1(p.vr + row0 + r) : 0.f;
#pragma unroll
            for (int f = 0; f < FPL; ++f) {
                const int col = col0 + tcol4(cl, f) * 4;
                if (col >= p.n) continue;
                float4 a;
                if (direct) {
                    a = a4(p.A + (int64_t)(row0 + r) * p.lda + col);   // inside lda (lda % 4 == 0)
                    if (col + 1 >= p.n) a.y = 0.f;                              // padding past n
                    if (col + 2 >= p.n) a.z = 0.f;
                    if (col + 3 >= p.n) a.w = 0.f;
                } else {
                    a = reinterpret_cast<const float4*>(stage)[r * CW + tcol4(cl, f)];
                }
                accumulate(k, f, a, xv[f], rv);
            }
        }
    }

    __device__ __forceinline__ void accumulate(int k, int f, const float4& a, const float4& xv, float rv) {
        if (DO_ROW) racc[k] += a.x * xv.x + a.y * xv.y + a.z * xv.z + a.w * xv.w;
        if (DO_COL) {
            cacc[f].x += a.x * rv; cacc[f].y += a.y * rv;
            cacc[f].z += a.z * rv; cacc[f].w += a.w * rv;
        }
    }

    __device__ __forceinline__ void finish(int ctid) {
        if (DO_ROW && cur_ti >= 0) flush_row(ctid);
        if (DO_COL && cur_tj >= 0) flush_col(ctid);
    }
};

}  // namespace cc
