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
//   * the A tile (streamed, no reuse) is staged by the producer warp with one
//     bulk async copy per tile row straight into shared memory (UBLKCP; it
//     never touches L1, the B200 form of the paper's bypass §4.3(II));
//   * the vc / vr slices -- the inter-CTA shared data -- are read by the
//     consumers with L1-allocating loads, so tasks of one SM that share bx (vc)
//     or by (vr) hit L1;
//   * partial out_r (out_c) sums are carried in registers across consecutive
//     tasks of one agent with the same by (bx) and flushed to L2 with one
//     (vector) RED only when the row (column) changes -- temporal inter-CTA
//     reuse kept on chip.  Under the default backend every CTA is a fresh task,
//     so it flushes every time: same code, no clustering.
// Consumers: 256 threads; CT = TC/4 threads cover one tile row with float4,
// RG = 256/CT row groups, each thread owns RPT = TR/RG rows.
#pragma once
#include "cc_mem.cuh"
#include "cc_runtime.cuh"

namespace cc {

struct GemvParams {
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
    static constexpr int kDefaultStages = TC >= 256 ? 4 : 3;
    static constexpr int kDefaultBatch = TC >= 256 ? 2 : 1;
    static constexpr int CT = TC / 4;
    static constexpr int RG = kConsumers / CT;
    static constexpr int RPT = TR / RG;
    static_assert(TC % 4 == 0 && kConsumers % CT == 0 && TR % RG == 0 && TR <= 32, "tile/thread shape");
    static_assert(CT <= 32 || CT % 32 == 0, "row group must be whole warps or a warp slice");
    static constexpr int WPR = CT > 32 ? CT / 32 : 1;   // warps per row group
    using Params = GemvParams;

    GemvParams p;
    int32_t cur_ti, cur_tj;
    float racc[RPT];
    float4 cacc;

    __device__ __forceinline__ explicit GemvBody(const GemvParams& prm) : p(prm), cur_ti(-1), cur_tj(-1) {
#pragma unroll
        for (int k = 0; k < RPT; ++k) racc[k] = 0.f;
        cacc = f4_zero();
    }

    // ---- producer: one bulk copy per tile row (rows past m are not copied)
    __device__ __forceinline__ void produce(const Sched&, int32_t bx, int32_t by, uint8_t* stage, uint64_t* full, int lane) {
        const int col0 = bx * TC;
        const int cols = p.n - col0 < TC ? p.n - col0 : TC;
        const uint32_t bytes = (uint32_t)((cols * 4 + 15) & ~15);    // within lda (lda % 4 == 0)
        const int row0 = by * TR;
        const int nrows = p.m - row0 < TR ? p.m - row0 : TR;
        stage_commit(full, lane, bytes * (uint32_t)nrows);
        if (lane < nrows)
            bulk_g2s(stage + lane * (TC * 4), p.A + (int64_t)(row0 + lane) * p.lda + col0, bytes, full);
    }

    // ---- ROW flush: sum racc over the CT threads of a row group, one RED per row
    __device__ __forceinline__ void flush_row(int ctid) {
        __shared__ float s_part[DO_ROW && WPR > 1 ? WPR : 1][DO_ROW && WPR > 1 ? TR : 1];
        const int cg = ctid % CT, rg = ctid / CT, lane = ctid & 31;
        constexpr int W = CT < 32 ? CT : 32;
#pragma unroll
        for (int k = 0; k < RPT; ++k) {
            float v = racc[k];
#pragma unroll
            for (int o = W / 2; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o, W);
            racc[k] = v;
        }
        const int row0 = cur_ti * TR;
        if constexpr (WPR == 1) {
            if (cg == 0) {
#pragma unroll
                for (int k = 0; k < RPT; ++k) {
                    int row = row0 + rg + k * RG;
                    if (row < p.m) red_add(p.out_r + row, racc[k]);
                }
            }
        } else {
            if (lane == 0) {
#pragma unroll
                for (int k = 0; k < RPT; ++k) s_part[cg / 32][rg + k * RG] = racc[k];
            }
            consumer_sync<kConsumers>();
            if (ctid < TR) {
                float v = 0.f;
#pragma unroll
                for (int w = 0; w < WPR; ++w) v += s_part[w][ctid];
                int row = row0 + ctid;
                if (row < p.m) red_add(p.out_r + row, v);
            }
            consumer_sync<kConsumers>();
        }
#pragma unroll
        for (int k = 0; k < RPT; ++k) racc[k] = 0.f;
    }

    // ---- COL flush: sum cacc over the RG row groups, one vector RED per 4 columns
    __device__ __forceinline__ void flush_col(int ctid) {
        const int cg = ctid % CT, rg = ctid / CT;
        const int col = cur_tj * TC + cg * 4;
        float4 v = cacc;
        if constexpr (RG > 1) {
            __shared__ float4 s_col[DO_COL ? RG : 1][DO_COL ? CT : 1];
            s_col[rg][cg] = cacc;
            consumer_sync<kConsumers>();
            if (ctid < CT) {
                v = s_col[0][ctid];
#pragma unroll
                for (int g = 1; g < RG; ++g) {
                    float4 u = s_col[g][ctid];
                    v.x += u.x; v.y += u.y; v.z += u.z; v.w += u.w;
                }
            }
            consumer_sync<kConsumers>();
        }
        if (ctid < CT && col < p.n) {
            if (col + 4 <= p.n) red_add4(p.out_c + col, v);
            else {
                red_add(p.out_c + col, v.x);
                if (col + 1 < p.n) red_add(p.out_c + col + 1, v.y);
                if (col + 2 < p.n) red_add(p.out_c + col + 2, v.z);
            }
        }
        cacc = f4_zero();
    }

    // ---- consumers: one logical CTA from the staged tile
    __device__ __forceinline__ void consume(int32_t bx, int32_t by, const uint8_t* stage, int ctid) {
        if (DO_ROW && by != cur_ti) { if (cur_ti >= 0) flush_row(ctid); cur_ti = by; }
        if (DO_COL && bx != cur_tj) { if (cur_tj >= 0) flush_col(ctid); cur_tj = bx; }
        const int cg = ctid % CT, rg = ctid / CT;
        const int col = bx * TC + cg * 4;
        const int rowb = by * TR + rg;
        if (col >= p.n) return;
        float4 xv = f4_zero();
        if (DO_ROW) {
            if (col + 4 <= p.n) xv = ld_cached4(p.vc + col);
            else {
                xv.x = ld_cached(p.vc + col);
                if (col + 1 < p.n) xv.y = ld_cached(p.vc + col + 1);
                if (col + 2 < p.n) xv.z = ld_cached(p.vc + col + 2);
            }
        }
        float rv[RPT];
        if (DO_COL) {
#pragma unroll
            for (int k = 0; k < RPT; ++k) {
                int row = rowb + k * RG;
                rv[k] = row < p.m ? ld_cached(p.vr + row) : 0.f;
            }
        }
        const float4* tile = reinterpret_cast<const float4*>(stage);
        const bool ragged = col + 4 > p.n;
#pragma unroll
        for (int k = 0; k < RPT; ++k) {
            const int r = rg + k * RG;
            if (rowb + k * RG >= p.m) break;
            float4 a = tile[r * CT + cg];
            if (ragged) {                                // lanes past n hold padding
                if (col + 1 >= p.n) a.y = 0.f;
                if (col + 2 >= p.n) a.z = 0.f;
                a.w = 0.f;
            }
            if (DO_ROW) racc[k] += a.x * xv.x + a.y * xv.y + a.z * xv.z + a.w * xv.w;
            if (DO_COL) {
                cacc.x += a.x * rv[k]; cacc.y += a.y * rv[k];
                cacc.z += a.z * rv[k]; cacc.w += a.w * rv[k];
            }
        }
    }

    __device__ __forceinline__ void finish(int ctid) {
        if (DO_ROW && cur_ti >= 0) flush_row(ctid);
        if (DO_COL && cur_tj >= 0) flush_col(ctid);
    }
};

}  // namespace cc
