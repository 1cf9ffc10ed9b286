// k_gemv.cuh -- tile body shared by the tiled matvec and ATAX / BICG / MVT.
//
// Logical CTA (bx, by) owns the TR x TC tile A[TR*by .., TC*bx ..] of a
// row-major fp32 matrix (Listing 2 layout: bx indexes the input
// vector B[idx], by the output C[idy]).  It contributes
//   ROW product:  out_r[rows of by] += A_tile   . vc[cols of bx]   (A x)
//   COL product:  out_c[cols of bx] += A_tile^T . vr[rows of by]   (A^T y)
// This is the cache-line-related class of Table 2 (ATX/MVT/BC).
//
// Where inter-CTA reuse is caught (the point of clustering):
//   * the vc / vr slices are read with L1-allocating loads, so consecutive or
//     concurrent tasks of one SM that share bx (vc) or by (vr) hit L1;
//   * the partial out_r (out_c) sums are carried in registers across
//     consecutive tasks of one agent with the same by (bx) and flushed to L2
//     with one vector RED only when the row (column) changes -- temporal
//     inter-CTA reuse kept on chip.  Under the default backend every CTA is a
//     fresh task, so it flushes every time: same code, no clustering.
//   * the A tile is streamed with L1::no_allocate so it cannot evict them.
// 256 threads: CT = TC/4 threads cover one tile row with float4, RG = 256/CT
// row groups, each thread owns RPT = TR/RG rows.
#pragma once
#include "cc_mem.cuh"

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
    static constexpr int kThreads = 256;
    static constexpr int CT = TC / 4;
    static constexpr int RG = kThreads / CT;
    static constexpr int RPT = TR / RG;
    static_assert(TC % 4 == 0 && kThreads % CT == 0 && TR % RG == 0, "tile/thread shape");
    static_assert(CT <= 32 || CT % 32 == 0, "row group must be whole warps or a warp slice");
    static constexpr int WPR = CT > 32 ? CT / 32 : 1;   // warps per row group
    using Params = GemvParams;

    GemvParams p;
    int32_t cur_ti, cur_tj;
    float racc[RPT];
    float4 cacc;
    int32_t cg, rg;

    __device__ __forceinline__ explicit GemvBody(const GemvParams& prm) : p(prm), cur_ti(-1), cur_tj(-1) {
        cg = threadIdx.x % CT;
        rg = threadIdx.x / CT;
#pragma unroll
        for (int k = 0; k < RPT; ++k) racc[k] = 0.f;
        cacc = f4_zero();
    }

    // ROW flush: sum racc over the CT threads of a row group, one RED per row.
    __device__ __forceinline__ void flush_row() {
        __shared__ float s_part[DO_ROW && WPR > 1 ? WPR : 1][DO_ROW && WPR > 1 ? TR : 1];
        const int lane = threadIdx.x & 31;
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
            const int wsub = cg / 32;   // which warp of the row group
            if (lane == 0) {
#pragma unroll
                for (int k = 0; k < RPT; ++k) s_part[wsub][rg + k * RG] = racc[k];
            }
            __syncthreads();
            if (threadIdx.x < TR) {
                float v = 0.f;
#pragma unroll
                for (int w = 0; w < WPR; ++w) v += s_part[w][threadIdx.x];
                int row = row0 + threadIdx.x;
                if (row < p.m) red_add(p.out_r + row, v);
            }
            __syncthreads();
        }
#pragma unroll
        for (int k = 0; k < RPT; ++k) racc[k] = 0.f;
    }

    // COL flush: sum cacc over the RG row groups, one vector RED per 4 columns.
    __device__ __forceinline__ void flush_col() {
        const int col = cur_tj * TC + cg * 4;
        float4 v = cacc;
        if constexpr (RG > 1) {
            __shared__ float4 s_col[DO_COL ? RG : 1][DO_COL ? CT : 1];
            s_col[rg][cg] = cacc;
            __syncthreads();
            if (threadIdx.x < CT) {
                v = s_col[0][threadIdx.x];
#pragma unroll
                for (int g = 1; g < RG; ++g) {
                    float4 u = s_col[g][threadIdx.x];
                    v.x += u.x; v.y += u.y; v.z += u.z; v.w += u.w;
                }
            }
            __syncthreads();
        }
        if (threadIdx.x < CT && col < p.n) {
            if (col + 4 <= p.n) red_add4(p.out_c + col, v);
            else {
                red_add(p.out_c + col, v.x);
                if (col + 1 < p.n) red_add(p.out_c + col + 1, v.y);
                if (col + 2 < p.n) red_add(p.out_c + col + 2, v.z);
            }
        }
        cacc = f4_zero();
    }

    __device__ __forceinline__ void run(int32_t bx, int32_t by) {
        if (DO_ROW && by != cur_ti) { if (cur_ti >= 0) flush_row(); cur_ti = by; }
        if (DO_COL && bx != cur_tj) { if (cur_tj >= 0) flush_col(); cur_tj = bx; }
        const int col = bx * TC + cg * 4;
        const int rowb = by * TR + rg;
        const bool col_ok = col < p.n;
        float4 a[RPT];
#pragma unroll
        for (int k = 0; k < RPT; ++k) {
            int row = rowb + k * RG;
            a[k] = (col_ok && row < p.m) ? ld_stream4(p.A + (int64_t)row * p.lda + col) : f4_zero();
        }
        float4 xv = f4_zero();
        if (DO_ROW && col_ok) {
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
        if (col_ok && col + 4 > p.n) {   // ragged right edge: drop lanes past n
#pragma unroll
            for (int k = 0; k < RPT; ++k) {
                if (col + 1 >= p.n) a[k].y = 0.f;
                if (col + 2 >= p.n) a[k].z = 0.f;
                a[k].w = 0.f;
            }
        }
#pragma unroll
        for (int k = 0; k < RPT; ++k) {
            if (DO_ROW) racc[k] += a[k].x * xv.x + a[k].y * xv.y + a[k].z * xv.z + a[k].w * xv.w;
            if (DO_COL) {
                cacc.x += a[k].x * rv[k]; cacc.y += a[k].y * rv[k];
                cacc.z += a[k].z * rv[k]; cacc.w += a[k].w * rv[k];
            }
        }
    }

    __device__ __forceinline__ void prefetch_l2(int32_t bx, int32_t by) {
        const int col0 = bx * TC;
        if (col0 >= p.n) return;
        int cols = p.n - col0 < TC ? p.n - col0 : TC;
        uint32_t bytes = (uint32_t)((cols * 4 + 15) & ~15);
        for (int k = 0; k < TR; ++k) {
            int row = by * TR + k;
            if (row >= p.m) break;
            prefetch_l2_bulk(p.A + (int64_t)row * p.lda + col0, bytes);
        }
    }

    __device__ __forceinline__ void finish() {
        if (DO_ROW && cur_ti >= 0) flush_row();
        if (DO_COL && cur_tj >= 0) flush_col();
    }
};

}  // namespace cc
