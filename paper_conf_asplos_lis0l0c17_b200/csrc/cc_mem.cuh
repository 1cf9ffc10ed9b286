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
    // not volatile: a pure read of data no one writes during the kernel, so the
    // compiler may hoist and batch these loads
    float4 v;
    asm("ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%0,%1,%2,%3}, [%4];"
        : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
// Same load as a volatile asm: volatile asm statements keep their program order,
// so a run of these issued back to back stays batched (all in flight at once)
// instead of being sunk next to their consumers by the scheduler.
__device__ __forceinline__ float4 ld_stream4_batched(const float* p) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
// Four streaming 16-byte loads issued by one asm statement: they leave the SM
// back to back whatever the scheduler does with their consumers.
__device__ __forceinline__ void ld_stream4_x4(float4& a, float4& b, float4& c, float4& d,
                                              const float* pa, const float* pb, const float* pc, const float* pd) {
    asm volatile(
        "ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%0,%1,%2,%3}, [%16];\n\t"
        "ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%4,%5,%6,%7}, [%17];\n\t"
        "ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%8,%9,%10,%11}, [%18];\n\t"
        "ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%12,%13,%14,%15}, [%19];"
        : "=f"(a.x), "=f"(a.y), "=f"(a.z), "=f"(a.w), "=f"(b.x), "=f"(b.y), "=f"(b.z), "=f"(b.w),
          "=f"(c.x), "=f"(c.y), "=f"(c.z), "=f"(c.w), "=f"(d.x), "=f"(d.y), "=f"(d.z), "=f"(d.w)
        : "l"(pa), "l"(pb), "l"(pc), "l"(pd));
}
// Eight of them in one statement (the 32 x 256 gemv tile: 4 rows x 2 float4 per lane).
__device__ __forceinline__ void ld_stream4_x8(float4* v, const float* const* p) {
    asm volatile(
        "ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%0,%1,%2,%3}, [%32];\n\t"
        "ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%4,%5,%6,%7}, [%33];\n\t"
        "ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%8,%9,%10,%11}, [%34];\n\t"
        "ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%12,%13,%14,%15}, [%35];\n\t"
        "ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%16,%17,%18,%19}, [%36];\n\t"
        "ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%20,%21,%22,%23}, [%37];\n\t"
        "ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%24,%25,%26,%27}, [%38];\n\t"
        "ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%28,%29,%30,%31}, [%39];"
        : "=f"(v[0].x), "=f"(v[0].y), "=f"(v[0].z), "=f"(v[0].w), "=f"(v[1].x), "=f"(v[1].y), "=f"(v[1].z), "=f"(v[1].w),
          "=f"(v[2].x), "=f"(v[2].y), "=f"(v[2].z), "=f"(v[2].w), "=f"(v[3].x), "=f"(v[3].y), "=f"(v[3].z), "=f"(v[3].w),
          "=f"(v[4].x), "=f"(v[4].y), "=f"(v[4].z), "=f"(v[4].w), "=f"(v[5].x), "=f"(v[5].y), "=f"(v[5].z), "=f"(v[5].w),
          "=f"(v[6].x), "=f"(v[6].y), "=f"(v[6].z), "=f"(v[6].w), "=f"(v[7].x), "=f"(v[7].y), "=f"(v[7].z), "=f"(v[7].w)
        : "l"(p[0]), "l"(p[1]), "l"(p[2]), "l"(p[3]), "l"(p[4]), "l"(p[5]), "l"(p[6]), "l"(p[7]));
}
// ---- L2 eviction priority (S§8(f)2: the bypass idea moved to B200's L2).
// createpolicy builds a 64-bit policy; .L2::cache_hint attaches it to a
// load/store/TMA copy.  evict_first: lines of a streamed operand leave L2
// first; evict_last: lines of a reused operand (vector slices, halos, x)
// stay longest.
__device__ __forceinline__ uint64_t l2_evict_first() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t l2_evict_last() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ float4 ld_stream4_h(const float* p, uint64_t pol) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.L2::256B.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ void ld_stream4_x8_h(float4* v, const float* const* p, uint64_t pol) {
    asm volatile(
        "ld.global.nc.L1::no_allocate.L2::cache_hint.L2::256B.v4.f32 {%0,%1,%2,%3}, [%32], %40;\n\t"
        "ld.global.nc.L1::no_allocate.L2::cache_hint.L2::256B.v4.f32 {%4,%5,%6,%7}, [%33], %40;\n\t"
        "ld.global.nc.L1::no_allocate.L2::cache_hint.L2::256B.v4.f32 {%8,%9,%10,%11}, [%34], %40;\n\t"
        "ld.global.nc.L1::no_allocate.L2::cache_hint.L2::256B.v4.f32 {%12,%13,%14,%15}, [%35], %40;\n\t"
        "ld.global.nc.L1::no_allocate.L2::cache_hint.L2::256B.v4.f32 {%16,%17,%18,%19}, [%36], %40;\n\t"
        "ld.global.nc.L1::no_allocate.L2::cache_hint.L2::256B.v4.f32 {%20,%21,%22,%23}, [%37], %40;\n\t"
        "ld.global.nc.L1::no_allocate.L2::cache_hint.L2::256B.v4.f32 {%24,%25,%26,%27}, [%38], %40;\n\t"
        "ld.global.nc.L1::no_allocate.L2::cache_hint.L2::256B.v4.f32 {%28,%29,%30,%31}, [%39], %40;"
        : "=f"(v[0].x), "=f"(v[0].y), "=f"(v[0].z), "=f"(v[0].w), "=f"(v[1].x), "=f"(v[1].y), "=f"(v[1].z), "=f"(v[1].w),
          "=f"(v[2].x), "=f"(v[2].y), "=f"(v[2].z), "=f"(v[2].w), "=f"(v[3].x), "=f"(v[3].y), "=f"(v[3].z), "=f"(v[3].w),
          "=f"(v[4].x), "=f"(v[4].y), "=f"(v[4].z), "=f"(v[4].w), "=f"(v[5].x), "=f"(v[5].y), "=f"(v[5].z), "=f"(v[5].w),
          "=f"(v[6].x), "=f"(v[6].y), "=f"(v[6].z), "=f"(v[6].w), "=f"(v[7].x), "=f"(v[7].y), "=f"(v[7].z), "=f"(v[7].w)
        : "l"(p[0]), "l"(p[1]), "l"(p[2]), "l"(p[3]), "l"(p[4]), "l"(p[5]), "l"(p[6]), "l"(p[7]), "l"(pol));
}
__device__ __forceinline__ float4 ld_cached4_h(const float* p, uint64_t pol) {
    float4 v;
    asm("ld.global.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
        : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ float ld_cached_h(const float* p, uint64_t pol) {
    float v;
    asm("ld.global.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ void st4_h(float* p, float4 v, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.v4.f32 [%0], {%1,%2,%3,%4}, %5;"
                 :: "l"(p), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w), "l"(pol) : "memory");
}
__device__ __forceinline__ void st1_h(float* p, float v, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.f32 [%0], %1, %2;" :: "l"(p), "f"(v), "l"(pol) : "memory");
}

// Default-cached load (allocates in L1): operands that other CTAs of the same
// cluster re-read (vector slices, halos).
__device__ __forceinline__ float4 ld_cached4(const float* p) {
    return *reinterpret_cast<const float4*>(p);
}
__device__ __forceinline__ float ld_cached(const float* p) { return *p; }
// Issue-ordered forms for gathers: volatile asm keeps program order, so a run
// of them leaves the SM back to back (all in flight) before any result is
// used -- the compiler otherwise interleaves each gather with its consumer.
__device__ __forceinline__ float ld_cached_issue(const float* p) {
    float v;
    asm volatile("ld.global.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}
// x gather that skips L1 (cached in L2 only): one L2 request per lane with no
// L1 tag lookup or fill
__device__ __forceinline__ float ld_l2only_issue(const float* p) {
    float v;
    asm volatile("ld.global.cg.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}
// hub values of the SpMV hub-column form: allocate in L1 and keep (evict_last)
__device__ __forceinline__ float ld_hot_issue(const float* p) {
    float v;
    asm volatile("ld.global.nc.L1::evict_last.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ int32_t ld_stream_i32_issue(const int32_t* p) {
    int32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ float ld_stream_f32_issue(const float* p) {
    float v;
    asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}

__device__ __forceinline__ float ld_stream_f32_h(const float* p, uint64_t pol) {
    float v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ int32_t ld_stream_i32_h(const int32_t* p, uint64_t pol) {
    int32_t v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
// Scalar streaming loads (read once; do not displace reused lines from L1).
__device__ __forceinline__ float ld_stream_f32(const float* p) {
    float v;
    asm("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ int32_t ld_stream_i32(const int32_t* p) {
    int32_t v;
    asm("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}

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
