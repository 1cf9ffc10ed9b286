// cc_mem.cuh -- memory-access helpers (sm_100a PTX).
#pragma once
#include <stdint.h>
#include <cuda.h>            // CUtensorMap
#include <cuda_runtime.h>

namespace cc {

// Streaming load that does not allocate in L1 (the B200 form of the paper's
// bypass, §4.3(II): ld.global.cg is a *strong* load on sm_100a,
// L1::no_allocate is the cheap bypass -> LDG.E.NA).  Used for operands with no
// inter-CTA reuse so they do not evict the reused slices.
__device__ __forceinline__ float4 ld_stream4(const float* p) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
// Default-cached load (allocates in L1): operands that other CTAs of the same
// cluster re-read (vector slices, halos).
__device__ __forceinline__ float4 ld_cached4(const float* p) {
    return *reinterpret_cast<const float4*>(p);
}
__device__ __forceinline__ float ld_cached(const float* p) { return *p; }

// Bulk L2 prefetch of `bytes` (multiple of 16, 16-byte aligned) at p
// (cp.async.bulk.prefetch.L2 -> UBLKPF.L2), the B200 form of PREFETCH_L1
// (Listing 5 l.34-37).
__device__ __forceinline__ void prefetch_l2_bulk(const void* p, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(p), "r"(bytes) : "memory");
}

// fire-and-forget fp32 reductions into L2 (RED), vector form where aligned
__device__ __forceinline__ void red_add(float* p, float v) {
    asm volatile("red.relaxed.gpu.global.add.f32 [%0], %1;" :: "l"(p), "f"(v) : "memory");
}
__device__ __forceinline__ void red_add4(float* p, float4 v) {
    asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1,%2,%3,%4};"
                 :: "l"(p), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w) : "memory");
}

__device__ __forceinline__ float4 f4_zero() { return make_float4(0.f, 0.f, 0.f, 0.f); }

}  // namespace cc
