// k_stencil.cuh -- 5-point Jacobi and 2D cross-correlation tile bodies.
//
// Logical CTA (bx, by) computes the 32 x 32 output tile at rows 32*by..,
// columns 32*bx.. .  The inter-CTA reuse is the halo: rows above/below and
// the columns left/right of a tile are the border data of its four neighbours
// (the cache-line/algorithm-related classes).  Halo and centre loads
// allocate in L1, so when clustering runs neighbouring tiles on the same SM
// close together (TILE order, Fig. 7) the halo comes from L1 instead of L2.
// 256 threads: thread (r = tid/8, c4 = tid%8) owns the float4 at row r,
// columns 4*c4 .. 4*c4+3 of the tile.
#pragma once
#include "cc_mem.cuh"

namespace cc {

// ---------------------------------------------------------------------------
// Jacobi 5-point sweep (reading R14, PolyBench jacobi-2d form):
//   b[i][j] = 0.2f * ((((c + w) + e) + n) + s)     on the interior,
//   b[i][j] = a[i][j]                               on the boundary.
// fp32, summed in that fixed order with no contraction, so the sweep is
// bit-reproducible against oracle_jacobi5_f32.
// ---------------------------------------------------------------------------
struct JacobiParams { const float* a; float* b; int64_t ld; int32_t rows, cols; };

struct Jacobi5Body {
    static constexpr int kThreads = 256;
    using Params = JacobiParams;
    JacobiParams p;
    __device__ __forceinline__ explicit Jacobi5Body(const JacobiParams& prm) : p(prm) {}

    __device__ __forceinline__ void run(int32_t bx, int32_t by) {
        __shared__ float4 tile[34][8];
        const int r = threadIdx.x >> 3, c4 = threadIdx.x & 7;
        const int x0 = bx * 32, y0 = by * 32;
        const int gy = y0 + r, gx = x0 + 4 * c4;
        const bool in_row = gy < p.rows, in_col = gx < p.cols;
        const float* a = p.a;
        float4 c = (in_row && in_col) ? ld_cached4(a + (int64_t)gy * p.ld + gx) : f4_zero();
        float4 up_h = f4_zero(), dn_h = f4_zero();
        if (r == 0 && y0 > 0 && in_col) up_h = ld_cached4(a + (int64_t)(y0 - 1) * p.ld + gx);
        if (r == 31 && y0 + 32 < p.rows && in_col) dn_h = ld_cached4(a + (int64_t)(y0 + 32) * p.ld + gx);
        float left = 0.f, right = 0.f;
        if (c4 == 0 && x0 > 0 && in_row) left = ld_cached(a + (int64_t)gy * p.ld + x0 - 1);
        if (c4 == 7 && x0 + 32 < p.cols && in_row) right = ld_cached(a + (int64_t)gy * p.ld + x0 + 32);
        tile[r + 1][c4] = c;
        if (r == 0) tile[0][c4] = up_h;
        if (r == 31) tile[33][c4] = dn_h;
        __syncthreads();
        const float4 up = tile[r][c4], dn = tile[r + 2][c4];
        float lw = __shfl_up_sync(0xffffffffu, c.w, 1, 8);
        float re = __shfl_down_sync(0xffffffffu, c.x, 1, 8);
        if (c4 == 0) lw = left;
        if (c4 == 7) re = right;
        if (!(in_row && in_col)) return;   // after the barrier and the shuffles
        float4 o;
        o.x = __fmul_rn(0.2f, __fadd_rn(__fadd_rn(__fadd_rn(__fadd_rn(c.x, lw), c.y), up.x), dn.x));
        o.y = __fmul_rn(0.2f, __fadd_rn(__fadd_rn(__fadd_rn(__fadd_rn(c.y, c.x), c.z), up.y), dn.y));
        o.z = __fmul_rn(0.2f, __fadd_rn(__fadd_rn(__fadd_rn(__fadd_rn(c.z, c.y), c.w), up.z), dn.z));
        o.w = __fmul_rn(0.2f, __fadd_rn(__fadd_rn(__fadd_rn(__fadd_rn(c.w, c.z), re), up.w), dn.w));
        const bool row_bd = (gy == 0) || (gy == p.rows - 1);
        const int cl = p.cols - 1;
        if (row_bd || gx == 0 || gx == cl) o.x = c.x;
        if (row_bd || gx + 1 == cl) o.y = c.y;
        if (row_bd || gx + 2 == cl) o.z = c.z;
        if (row_bd || gx + 3 == cl) o.w = c.w;
        float* dst = p.b + (int64_t)gy * p.ld + gx;
        if (gx + 4 <= p.cols) *reinterpret_cast<float4*>(dst) = o;
        else {
            dst[0] = o.x;
            if (gx + 1 < p.cols) dst[1] = o.y;
            if (gx + 2 < p.cols) dst[2] = o.z;
        }
    }
    __device__ __forceinline__ void prefetch_l2(int32_t bx, int32_t by) {
        const int x0 = bx * 32;
        if (x0 >= p.cols) return;
        int cols = p.cols - x0 < 32 ? p.cols - x0 : 32;
        uint32_t bytes = (uint32_t)((cols * 4 + 15) & ~15);
        for (int k = -1; k <= 32; ++k) {
            int row = by * 32 + k;
            if (row < 0) continue;
            if (row >= p.rows) break;
            prefetch_l2_bulk(p.a + (int64_t)row * p.ld + x0, bytes);
        }
    }
    __device__ __forceinline__ void finish() {}
};

// ---------------------------------------------------------------------------
// 2D cross-correlation with a (2R+1)^2 filter (reading R15):
//   out[i][j] = sum_{a,b} w[a+R][b+R] * in[i+a][j+b]   interior, else 0.
// The input tile plus an R halo is staged in shared memory with aligned
// float4 loads covering columns x0-4 .. x0+35.
// ---------------------------------------------------------------------------
template <int R>
struct ConvParams { const float* in; float* out; int64_t ld; int32_t rows, cols; float w[(2 * R + 1) * (2 * R + 1)]; };

template <int R>
struct Conv2dBody {
    static constexpr int kThreads = 256;
    static constexpr int K = 2 * R + 1;
    static constexpr int SR = 32 + 2 * R;   // staged rows
    using Params = ConvParams<R>;
    ConvParams<R> p;   // filter lives in the parameter bank (constant operands)
    __device__ __forceinline__ explicit Conv2dBody(const ConvParams<R>& prm) : p(prm) {}

    __device__ __forceinline__ void run(int32_t bx, int32_t by) {
        __shared__ float4 s_in[SR][10];
        const int x0 = bx * 32, y0 = by * 32;
        for (int idx = threadIdx.x; idx < SR * 10; idx += kThreads) {
            const int rr = idx / 10, cc = idx - rr * 10;
            const int gy = y0 - R + rr, gx = x0 - 4 + 4 * cc;
            float4 v = f4_zero();
            if (gy >= 0 && gy < p.rows && gx >= 0 && gx < p.cols) v = ld_cached4(p.in + (int64_t)gy * p.ld + gx);
            s_in[rr][cc] = v;
        }
        __syncthreads();
        const int r = threadIdx.x >> 3, c4 = threadIdx.x & 7;
        const int gy = y0 + r, gx = x0 + 4 * c4;
        float acc[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
        for (int dy = 0; dy < K; ++dy) {
            const float4* row = &s_in[r + dy][c4];
            float4 q0 = row[0], q1 = row[1], q2 = row[2];
            const float win[12] = {q0.x, q0.y, q0.z, q0.w, q1.x, q1.y, q1.z, q1.w, q2.x, q2.y, q2.z, q2.w};
#pragma unroll
            for (int dx = 0; dx < K; ++dx) {
                const float wt = p.w[dy * K + dx];
#pragma unroll
                for (int e = 0; e < 4; ++e) acc[e] = fmaf(wt, win[4 + e + dx - R], acc[e]);
            }
        }
        if (gy >= p.rows || gx >= p.cols) return;
        const bool row_in = gy >= R && gy < p.rows - R;
        float4 o;
        o.x = (row_in && gx + 0 >= R && gx + 0 < p.cols - R) ? acc[0] : 0.f;
        o.y = (row_in && gx + 1 >= R && gx + 1 < p.cols - R) ? acc[1] : 0.f;
        o.z = (row_in && gx + 2 >= R && gx + 2 < p.cols - R) ? acc[2] : 0.f;
        o.w = (row_in && gx + 3 >= R && gx + 3 < p.cols - R) ? acc[3] : 0.f;
        float* dst = p.out + (int64_t)gy * p.ld + gx;
        if (gx + 4 <= p.cols) *reinterpret_cast<float4*>(dst) = o;
        else {
            dst[0] = o.x;
            if (gx + 1 < p.cols) dst[1] = o.y;
            if (gx + 2 < p.cols) dst[2] = o.z;
        }
    }
    __device__ __forceinline__ void prefetch_l2(int32_t bx, int32_t by) {
        const int x0 = bx * 32 - 4;
        int c0 = x0 < 0 ? 0 : x0;
        int c1 = bx * 32 + 36; if (c1 > p.cols) c1 = p.cols;
        if (c1 <= c0) return;
        uint32_t bytes = (uint32_t)(((c1 - c0) * 4 + 15) & ~15);
        for (int k = -R; k < 32 + R; ++k) {
            int row = by * 32 + k;
            if (row < 0) continue;
            if (row >= p.rows) break;
            prefetch_l2_bulk(p.in + (int64_t)row * p.ld + c0, bytes);
        }
    }
    __device__ __forceinline__ void finish() {}
};

}  // namespace cc
