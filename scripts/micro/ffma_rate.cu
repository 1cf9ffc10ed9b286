// FFMA issue-rate microbenchmark for sm_100a: which FFMA operand forms reach
// one warp instruction per clock per SM sub-partition (128 FMA/clk/SM)?
//   reg:   a = fma(x, w_reg, a)      (w in a register)
//   const: a = fma(x, p.w[k], a)     (w from the kernel parameter bank)
//   imm:   a = fma(x, 1.0001f, a)    (w an immediate)
// 16 independent accumulators per thread, 2048 FFMA per accumulator.
#include <cstdio>
#include <cuda_runtime.h>
struct W { float w[16]; };
template <int MODE>
__global__ void __launch_bounds__(256) k(const __grid_constant__ W p, float* out, float seed) {
    float a[16], x = seed + threadIdx.x * 1e-7f;
    float wr[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) { a[i] = i * 1e-3f; wr[i] = 0.999f + threadIdx.x * 1e-9f + i * 1e-6f; }
#pragma unroll 1
    for (int it = 0; it < 128; ++it) {
#pragma unroll
        for (int r = 0; r < 16; ++r)
#pragma unroll
            for (int i = 0; i < 16; ++i) {
                if (MODE == 0) a[i] = fmaf(x, wr[(i + r) & 15], a[i]);
                else if (MODE == 1) a[i] = fmaf(x, p.w[(i + r) & 15], a[i]);
                else a[i] = fmaf(x, 1.0001f, a[i]);
            }
    }
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < 16; ++i) s += a[i];
    if (s == 12345.f) out[0] = s;
}
int main() {
    int dev = 0, sms = 0, clk = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
    float* out; cudaMalloc(&out, 4);
    W p; for (int i = 0; i < 16; ++i) p.w[i] = 0.999f + i * 1e-6f;
    const char* names[3] = {"reg", "const", "imm"};
    for (int mode = 0; mode < 3; ++mode) {
        for (int bps = 4; bps <= 8; bps += 4) {
            dim3 grid(sms * bps * 4), block(256);
            cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
            for (int rep = 0; rep < 2; ++rep) {
                cudaEventRecord(a);
                if (mode == 0) k<0><<<grid, block>>>(p, out, 1.0f);
                else if (mode == 1) k<1><<<grid, block>>>(p, out, 1.0f);
                else k<2><<<grid, block>>>(p, out, 1.0f);
                cudaEventRecord(b); cudaEventSynchronize(b);
            }
            float ms; cudaEventElapsedTime(&ms, a, b);
            double fma = (double)grid.x * 256 * 128 * 16 * 16;
            double tf = 2 * fma / (ms * 1e-3) / 1e12;
            printf("%-6s blocks/SM-wave %d: %.3f ms  %.2f TFLOP/s  %.1f FMA/clk/SM at %d MHz\n", names[mode], bps,
                   ms, tf, fma / (ms * 1e-3) / sms / (clk * 1e3), clk / 1000);
        }
    }
    cudaError_t e = cudaGetLastError();
    printf("status: %s\n", cudaGetErrorString(e));
    return 0;
}
