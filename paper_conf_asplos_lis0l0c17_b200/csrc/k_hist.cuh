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
// One-shot CTAs (default order, redirection) count into per-warp shared-
// memory sub-histograms with shared atomics and add them to the 64 global
// counters per chunk.  Persistent agents (round 2) privatise further: every
// consumer lane owns 64 16-bit counters in the agent's persistent-only
// shared memory (layout [bin][lane], so a warp's 32 counters of one bin are
// 32 consecutive half-words: no bank conflict, no atomic -- a load, an add
// and a store per byte), kept across all the agent's tasks and reduced into
// the global counters every 256 tasks (before a 16-bit counter could wrap:
// a lane counts at most 128 bytes per task) and when the agent retires.
// The one-shot form cannot afford this: it would zero and reduce 16 K
// counters per 32 KiB chunk.
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
    static constexpr int kPersistentSmemBytes = 64 * kConsumers * 2;   // [bin][lane] uint16 counters
    static constexpr int kFlushTasks = 256;
    using Params = HistParams;
    const HistParams& p;
    int32_t l2h = 0;
    bool started = false;                       // sub-histograms zeroed (uniform over consumers)
    int32_t tasks = 0;                          // persistent path: tasks since the last flush
    uint16_t* priv_ = nullptr;                  // persistent path: this agent's lane counters
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

    // persistent path ------------------------------------------------------
    __device__ __forceinline__ static uint16_t* lane_counters(const Sched& s) {
        extern __shared__ uint8_t dyn_smem[];
        return reinterpret_cast<uint16_t*>(ring_base(dyn_smem) + (size_t)s.stages * s.stage_bytes);
    }
    __device__ __forceinline__ static void bump(uint16_t* c, uint32_t bin, int lane_id) {
        uint16_t* q = c + bin * kConsumers + lane_id;
        *q = (uint16_t)(*q + 1);
    }
    __device__ __forceinline__ static void count_word_priv(uint16_t* c, uint32_t w, int ctid) {
        bump(c, (w >> 2) & 63u, ctid);
        bump(c, (w >> 10) & 63u, ctid);
        bump(c, (w >> 18) & 63u, ctid);
        bump(c, (w >> 26) & 63u, ctid);
    }
    // every consumer: reduce the lane counters into the global counts and zero them
    __device__ __forceinline__ void flush_priv(uint16_t* c, int ctid) const {
        consumer_sync<kConsumers>();
        const int bin = ctid >> 2, q = ctid & 3;                    // 4 threads per bin, 64 lanes each
        uint4* row = reinterpret_cast<uint4*>(c + bin * kConsumers + q * 64);
        uint32_t v = 0;
#pragma unroll
        for (int k = 0; k < 8; ++k) {                               // 8 x 8 half-words
            const uint4 x = row[k];
            v += (x.x & 0xffffu) + (x.x >> 16) + (x.y & 0xffffu) + (x.y >> 16) + (x.z & 0xffffu) + (x.z >> 16) +
                 (x.w & 0xffffu) + (x.w >> 16);
            row[k] = make_uint4(0u, 0u, 0u, 0u);
        }
        v += __shfl_xor_sync(0xffffffffu, v, 1);
        v += __shfl_xor_sync(0xffffffffu, v, 2);
        if (q == 0 && v) atomicAdd(p.counts + bin, v);
        consumer_sync<kConsumers>();
    }

    __device__ __forceinline__ void consume(const Sched& s, int32_t bx, int32_t by, const uint8_t* stage, int ctid) {
        if (!s.oneshot) { consume_priv(s, bx, stage, ctid); return; }
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

    __device__ __forceinline__ void consume_priv(const Sched& s, int32_t bx, const uint8_t* stage, int ctid) {
        uint16_t* c = lane_counters(s);
        priv_ = c;
        if (!started) {
            uint4* z = reinterpret_cast<uint4*>(c);
            for (int i = ctid; i < kPersistentSmemBytes / 16; i += kConsumers) z[i] = make_uint4(0u, 0u, 0u, 0u);
            consumer_sync<kConsumers>();
            started = true;
        }
        const int64_t base = (int64_t)bx * HIST_CHUNK;
        const int64_t rem = p.n - base;
        const int len = rem < HIST_CHUNK ? (int)rem : HIST_CHUNK;
        const int nv = len >> 4;
        if (s.staging == 1) {
            const uint4* src = reinterpret_cast<const uint4*>(stage);
#pragma unroll 4
            for (int i = ctid; i < nv; i += kConsumers) {
                const uint4 w = src[i];
                count_word_priv(c, w.x, ctid); count_word_priv(c, w.y, ctid);
                count_word_priv(c, w.z, ctid); count_word_priv(c, w.w, ctid);
            }
        } else {
            const uint8_t* g = p.data + base;
#pragma unroll 4
            for (int i = ctid; i < nv; i += kConsumers) {
                const uint4 w = s.staging == 2 ? *reinterpret_cast<const uint4*>(g + 16 * i) : ld_stream_u4(g + 16 * i);
                count_word_priv(c, w.x, ctid); count_word_priv(c, w.y, ctid);
                count_word_priv(c, w.z, ctid); count_word_priv(c, w.w, ctid);
            }
        }
        const int tail = len - 16 * nv;
        if (ctid < tail) bump(c, p.data[base + 16 * nv + ctid] >> 2, ctid);
        if (++tasks == kFlushTasks) {
            flush_priv(c, ctid);
            tasks = 0;
        }
    }

    __device__ __forceinline__ void finish(int ctid) {
        if (!started) return;                                          // agent that ran no task
        if (priv_) { flush_priv(priv_, ctid); return; }
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
