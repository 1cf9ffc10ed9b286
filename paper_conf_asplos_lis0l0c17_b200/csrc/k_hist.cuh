// k_hist.cuh -- 64-bin histogram tile body (S§8(f)3).
//
// The paper's HST (Table 2: "histogram 64-bin histogramming", data-
// related) -- the CUDA SDK histogram64, reading R24:
//     counts[k] = #{ i : data[i] >> 2 == k },  k = 0..63.
// Its input is a pure stream (no inter-CTA reuse); its inter-CTA sharing is
// on the output: every CTA updates the same 64 counters.  It is the second
// workload class for the paper's claim that CTA prefetching with a reshaped
// order helps kernels without exploitable locality (section 4.3(III)).
//
// Logical CTA b owns the 32 KiB input chunk [32768 b, 32768 (b+1)).  The
// producer warp stages it with one 1D bulk copy (TMA) into the agent's ring
// -- the successor's chunk is in flight while the current one is counted,
// which is the prefetch the agent's ordered task stream makes possible.
// Consumers count into per-warp shared-memory sub-histograms with shared
// atomics.  A persistent agent keeps its sub-histograms across all its tasks
// and adds them to the 64 global counters once, when it retires (finish); a
// one-shot CTA (default order) does that per chunk.
#pragma once
#include "cc_mem.cuh"
#include "cc_runtime.cuh"

namespace cc {

struct HistParams { const uint8_t* data; int64_t n; uint32_t* counts; };

constexpr int HIST_CHUNK = 32768;               // input bytes per logical CTA
constexpr int HIST_WARPS = 8;

__device__ __forceinline__ uint4 ld_stream_u4(const void* p) {
    uint4 v;
    asm("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
        : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}

struct HistBody {
    static constexpr int kConsumers = HIST_WARPS * 32;
    static constexpr int kStageBytes = HIST_CHUNK;
    static constexpr int kDefaultStages = 3;
    static constexpr int kDefaultBatch = 2;
    static constexpr int kMinAgents = 2;
    static constexpr int kGroups = 1;
    using Params = HistParams;
    const HistParams& p;
    int32_t l2h = 0;
    bool started = false;                       // sub-histograms zeroed (uniform over consumers)
    __device__ __forceinline__ explicit HistBody(const HistParams& prm) : p(prm) {}

    __device__ __forceinline__ static uint32_t (&sub())[HIST_WARPS][64] {
        __shared__ uint32_t s_h[HIST_WARPS][64];
        return s_h;
    }

    __device__ __forceinline__ void produce(const Sched& s, int32_t bx, int32_t, uint8_t* stage, uint64_t* full, int lane) {
        if (s.staging != 1) { stage_commit(full, lane, 0); return; }   // L1 / direct: consumers load
        const int64_t base = (int64_t)bx * HIST_CHUNK;
        const int64_t rem = p.n - base;
        const uint32_t len = rem < HIST_CHUNK ? (uint32_t)rem : (uint32_t)HIST_CHUNK;
        const uint32_t bulk = len & ~15u;                              // the 16-byte multiple part
        stage_commit(full, lane, bulk);
        if (lane == 0 && bulk) bulk_g2s(stage, p.data + base, bulk, full);
    }

    __device__ __forceinline__ static void count_word(uint32_t (&h)[64], uint32_t w) {
        atomicAdd(&h[(w >> 2) & 63u], 1u);
        atomicAdd(&h[(w >> 10) & 63u], 1u);
        atomicAdd(&h[(w >> 18) & 63u], 1u);
        atomicAdd(&h[(w >> 26) & 63u], 1u);
    }

    __device__ __forceinline__ void consume(const Sched& s, int32_t bx, int32_t, const uint8_t* stage, int ctid) {
        auto& H = sub();
        if (!started) {
            for (int i = ctid; i < HIST_WARPS * 64; i += kConsumers) (&H[0][0])[i] = 0u;
            consumer_sync<kConsumers>();
            started = true;
        }
        uint32_t (&h)[64] = H[ctid >> 5];
        const int64_t base = (int64_t)bx * HIST_CHUNK;
        const int64_t rem = p.n - base;
        const int len = rem < HIST_CHUNK ? (int)rem : HIST_CHUNK;
        const int nv = len >> 4;
        if (s.staging == 1) {
            const uint4* src = reinterpret_cast<const uint4*>(stage);
#pragma unroll 4
            for (int i = ctid; i < nv; i += kConsumers) {
                const uint4 w = src[i];
                count_word(h, w.x); count_word(h, w.y); count_word(h, w.z); count_word(h, w.w);
            }
        } else {
            const uint8_t* g = p.data + base;
#pragma unroll 4
            for (int i = ctid; i < nv; i += kConsumers) {
                const uint4 w = s.staging == 2 ? *reinterpret_cast<const uint4*>(g + 16 * i) : ld_stream_u4(g + 16 * i);
                count_word(h, w.x); count_word(h, w.y); count_word(h, w.z); count_word(h, w.w);
            }
        }
        const int tail = len - 16 * nv;                                // < 16 bytes past the bulk part
        if (ctid < tail) atomicAdd(&h[p.data[base + 16 * nv + ctid] >> 2], 1u);
    }

    __device__ __forceinline__ void finish(int ctid) {
        if (!started) return;                                          // agent that ran no task
        auto& H = sub();
        consumer_sync<kConsumers>();
        if (ctid < 64) {
            uint32_t v = 0;
#pragma unroll
            for (int w = 0; w < HIST_WARPS; ++w) v += H[w][ctid];
            if (v) atomicAdd(p.counts + ctid, v);
        }
    }
};

}  // namespace cc
