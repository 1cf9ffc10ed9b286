// cc_runtime.cuh -- the agent runtime (binding + task loop) for sm_100a.
//
// PAPER.md §4.2.3 Step 3 "Binding", §4.2.4(2) agent-based
// clustering (Fig. 8(D), Listing 5), §4.3(I) CTA throttling
// and §4.3(III) prefetching.
//
// An agent is a persistent, warp-specialised CTA:
//   warp 0        scheduler/producer: binds the agent to its SM's cluster,
//                 pops logical-CTA slots ahead of use and stages each task's
//                 input tile into a ring of `stages` shared-memory buffers
//                 (bulk async copies / cp.async, completion on an mbarrier);
//   warps 1..8    consumers: run the original kernel body on each staged
//                 task in order, then release the buffer (empty mbarrier).
// The ring is the B200 form of Listing 5's "prefetch the next CTA" -- the
// next tasks' data is in flight while the current one computes -- and it makes
// the bytes in flight independent of how many agents are active, so
// throttling (active_agents) no longer starves the memory system.
//
// B200-first differences from Listing 5:
//   * cluster i binds to the SM of dense rank i from a probe-built table, not to
//     raw %smid (virtual, possibly sparse; reading R7);
//   * slots are popped in batches from a per-cluster queue with relaxed atomics
//     (the next batch's atomic is issued as soon as the current batch starts),
//     instead of a static stride v += ACTIVE_AGENTS; an agent whose queue is
//     empty steals, scanning all queues warp-parallel, so every logical CTA runs
//     exactly once whatever the hardware does with agent placement (R9/R10);
//   * no gpu-scope fence or acquire anywhere: on sm_100a those emit CCTL.IVALL,
//     which would wipe the very L1 contents clustering tries to keep;
//   * the workspace resets itself (last agent out), so a launch is one kernel.
#pragma once
#include <stdint.h>
#include <cuda_runtime.h>
#include "cc_index.cuh"

namespace cc {

enum : int32_t { MODE_AGENT = 0, MODE_IDENTITY = 1, MODE_STATIC = 2 };
constexpr int MAX_STAGES = 8;
constexpr int PRODUCER_THREADS = 32;

// Everything a task loop needs, passed by value as a kernel parameter.
struct Sched {
    Grid g;
    const int32_t* user;          // USER order table: v -> lin (device)
    const int32_t* rank_of_smid;  // %smid -> dense SM rank or -1 (device)
    int32_t smid_span;
    int32_t* ws;                  // workspace: agent_ctr[M+1] | head[M] | gq | done | claimed | chunk[M]
    int32_t mode;                 // MODE_AGENT / MODE_IDENTITY / MODE_STATIC
    int32_t active_agents;
    int32_t throttle;             // active_agents < agents launched per SM
    int32_t steal;
    int32_t stages;               // ring depth (agent backends; 1 for one-shot CTAs)
    int32_t batch;                // slots claimed per queue atomic
    uint32_t stage_bytes;         // bytes per ring buffer (128-byte multiple)
    int32_t staging;              // cc_staging: 1 TMA, 2 L1-allocating cp.async, 3 direct
    int32_t l2_hint;              // cc_l2_hint bits: 1 streamed operand evict_first, 2 reused operand evict_last
    uint32_t* census;             // optional outputs (see ctaclust.h)
    int32_t* exec_sm;
    int32_t* map;
};

__device__ __forceinline__ int32_t* ws_agent_ctr(const Sched& s) { return s.ws; }
__device__ __forceinline__ int32_t* ws_head(const Sched& s) { return s.ws + s.g.M + 1; }
__device__ __forceinline__ int32_t* ws_gq(const Sched& s) { return s.ws + 2 * s.g.M + 1; }
__device__ __forceinline__ int32_t* ws_done(const Sched& s) { return s.ws + 2 * s.g.M + 2; }
__device__ __forceinline__ int32_t* ws_claimed(const Sched& s) { return s.ws + 2 * s.g.M + 3; }
// chunk counters per cluster (warp-agent kernels, k_jwave.cuh), after the rest
__device__ __forceinline__ int32_t* ws_chunk(const Sched& s) { return s.ws + 2 * s.g.M + 4; }
inline size_t ws_ints(int32_t M) { return (size_t)(3 * M + 4); }

// ---------------------------------------------------------------------------
// PTX helpers
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smid() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t nsmid() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%nsmid;" : "=r"(r));
    return r;
}
__device__ __forceinline__ int32_t ld_relaxed(const int32_t* p) {
    int32_t v;
    asm volatile("ld.relaxed.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ int32_t atom_add_relaxed(int32_t* p, int32_t v) {
    int32_t old;
    asm volatile("atom.relaxed.gpu.global.add.s32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
    return old;
}
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}
// The suspend-time hint lets a waiting warp sleep in hardware until the phase
// completes (or the hint expires) instead of re-issuing try_wait: spinning
// consumer warps otherwise eat the issue slots the working warps need.
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n\t"
        "@!p bra WAIT_%=;\n}" :: "r"(smem_u32(bar)), "r"(parity), "r"(1000000u) : "memory");
}
// (Round 1 measured exponential nanosleep back-off and test_wait + timed
// sleep in place of the suspend-hint wait, for the producer and the
// consumers: slower or equal -- profiles/r05/diag, r07/diag.  Round 2
// re-measured a fixed 250-2000 ns producer sleep on the FP32-bound 7x7 conv,
// whose producer waits on `empty` 5 M times per launch (15 % of its issued
// instructions, ncu r10h): equal or up to 10 % slower, gpurun_out r10j.)
// 1D bulk async copy global -> shared, completion counted on `bar` (UBLKCP).
// dst, src 16-byte aligned, bytes a multiple of 16.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
// 16-byte cp.async that also allocates the line in L1 (.ca): the staged data
// doubles as L1-resident data for neighbouring tasks on the same SM.
// src_bytes < 16 zero-fills the rest (0 => pure zero fill, no read).
__device__ __forceinline__ void cp_async_ca16(void* dst, const void* src, uint32_t src_bytes) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 16, %2;"
                 :: "r"(smem_u32(dst)), "l"(src), "r"(src_bytes) : "memory");
}
// the bypassing variant (.cg: cached in L2 only)
__device__ __forceinline__ void cp_async_cg16(void* dst, const void* src, uint32_t src_bytes) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;"
                 :: "r"(smem_u32(dst)), "l"(src), "r"(src_bytes) : "memory");
}
// this thread's prior cp.async ops complete -> one (pre-counted) arrival on bar
__device__ __forceinline__ void cp_async_arrive(uint64_t* bar) {
    asm volatile("cp.async.mbarrier.arrive.shared::cta.b64 [%0];" :: "r"(smem_u32(bar)) : "memory");
}
// 2D TMA tile load (UTMALDG) of the box at (x, y) -- out-of-range elements are
// zero-filled -- completion counted on `bar` (the box's full byte count).
__device__ __forceinline__ void tma_load_2d(void* dst, const void* tmap, int32_t x, int32_t y, uint64_t* bar) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                 :: "r"(smem_u32(dst)), "l"(tmap), "r"(x), "r"(y), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void tma_load_2d_h(void* dst, const void* tmap, int32_t x, int32_t y, uint64_t* bar,
                                              uint64_t pol) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint"
                 " [%0], [%1, {%2, %3}], [%4], %5;"
                 :: "r"(smem_u32(dst)), "l"(tmap), "r"(x), "r"(y), "r"(smem_u32(bar)), "l"(pol) : "memory");
}
// L2 hint bits (cc_launch_opts.l2_hint)
enum : int32_t { L2H_STREAM_FIRST = 1, L2H_REUSE_LAST = 2, L2H_HALO_LAST = 4 };
// named barrier among the consumer warps only (the producer warp never joins)
// (barrier 1 + g for consumer group g of N threads; groups never share one)
template <int N>
__device__ __forceinline__ void consumer_sync() {
    // literal ids, so ptxas reserves only the barriers actually used
    switch ((int)(threadIdx.x - 32) / N) {
    case 0: asm volatile("bar.sync 1, %0;" :: "n"(N) : "memory"); break;
    case 1: asm volatile("bar.sync 2, %0;" :: "n"(N) : "memory"); break;
    case 2: asm volatile("bar.sync 3, %0;" :: "n"(N) : "memory"); break;
    default: asm volatile("bar.sync 4, %0;" :: "n"(N) : "memory"); break;
    }
}

// Stage protocol for Body::produce (warp 0, all lanes): the full barrier has
// an arrival count of 1.  Lanes may first issue cp.async + cp_async_arrive
// (each pre-counts itself), then call stage_commit(), which makes lane 0's
// single arrival carrying the byte count of the bulk copies issued after it.
__device__ __forceinline__ void stage_commit(uint64_t* full, int lane, uint32_t bulk_bytes) {
    __syncwarp();
    if (lane == 0) mbar_arrive_tx(full, bulk_bytes);
    __syncwarp();
}

__device__ __forceinline__ void lin_to_bxby(const Sched& s, int32_t v, int32_t* lin, int32_t* bx, int32_t* by) {
    if (s.mode == MODE_IDENTITY) {                       // row-major, ignores the plan's order
        *by = v / s.g.gx; *bx = v - *by * s.g.gx; *lin = v;
    } else if (s.g.order == ORDER_USER) {
        int32_t l = s.user[v];
        *by = l / s.g.gx; *bx = l - *by * s.g.gx; *lin = l;
    } else {
        decode(s.g, v, bx, by);
        *lin = *by * s.g.gx + *bx;
    }
}

// Producer-warp form (v warp-uniform, all 32 lanes present).  A USER order
// table lookup is a dependent L2 round trip per task on the scheduler's
// critical path (measured 2.3x slower conv 3x3 than the computed orders);
// the warp instead loads a window of 32 consecutive positions with one
// coalesced load into shared memory (win[0] = base, win[1..32] = entries;
// nothing held in registers across the task loop) and serves the cluster's
// consecutive pops from it.
__device__ __forceinline__ void lin_to_bxby_warp(const Sched& s, int32_t* win, int32_t v, int lane, int32_t* lin,
                                                 int32_t* bx, int32_t* by) {
    if (s.mode != MODE_IDENTITY && s.g.order == ORDER_USER) {
        const int32_t base = *(volatile int32_t*)win;
        if (v < base || v >= base + 32) {
            const int32_t u = v + lane < s.g.V ? s.user[v + lane] : 0;
            __syncwarp();
            win[1 + lane] = u;
            if (lane == 0) win[0] = v;
            __syncwarp();
        }
        const int32_t l = ((volatile int32_t*)win)[1 + v - *(volatile int32_t*)win];
        *by = l / s.g.gx; *bx = l - *by * s.g.gx; *lin = l;
    } else {
        lin_to_bxby(s, v, lin, bx, by);
    }
}

__device__ __forceinline__ void record(const Sched& s, int32_t v, int32_t lin) {
    if (s.census) atomicAdd(s.census + lin, 1u);
    if (s.exec_sm) s.exec_sm[lin] = (int32_t)smid();
    if (s.map) s.map[v] = lin;
}

// ---------------------------------------------------------------------------
// Scheduler (producer warp).  Lane 0 owns the queue state; the whole warp
// helps with the steal scan.
// ---------------------------------------------------------------------------
struct Prod {
    int32_t q;        // queue being drained (-1: none left)
    int32_t home;     // first queue, and where the steal scan starts
    int32_t bq, bw, be;   // current batch: slots [bw, be) of queue bq
    int32_t sq, sw;   // speculative claim in flight: raw fetch-add result on queue sq
    int32_t spec;
    int32_t mine;     // slots claimed since the last flush to the global `claimed` count
};

__device__ __forceinline__ int32_t q_size(const Sched& s, int32_t q) {
    return s.mode == MODE_IDENTITY ? s.g.V : cluster_size(s.g, q);
}
__device__ __forceinline__ int32_t q_start(const Sched& s, int32_t q) {
    return s.mode == MODE_IDENTITY ? 0 : cluster_start(s.g, q);
}
__device__ __forceinline__ int32_t* q_head(const Sched& s, int32_t q) {
    return s.mode == MODE_IDENTITY ? ws_gq(s) : ws_head(s) + q;
}

// Position of slot w of queue q.  (Draining odd clusters back to front was
// measured in round 1 -- +-1 % on the agents, 2-11 % slower static -- and dropped.)
__device__ __forceinline__ int32_t q_pos(const Sched& s, int32_t q, int32_t w) {
    return q_start(s, q) + w;
}

// lane 0 only.  Returns an order position, or -1 with *scan = 1 when the queue
// being drained is empty and a steal scan should follow, or -1 with *scan = 0
// when this agent is done.
__device__ __forceinline__ int32_t lane0_next(const Sched& s, Prod& P, int32_t* scan) {
    *scan = 0;
    if (P.bw < P.be) return q_pos(s, P.bq, P.bw++);
    for (;;) {
        int32_t sq, w;
        if (P.spec) { sq = P.sq; w = P.sw; P.spec = 0; }
        else if (P.q >= 0) { sq = P.q; w = atom_add_relaxed(q_head(s, sq), s.batch); }
        else return -1;
        const int32_t size = q_size(s, sq);
        if (w < size) {
            P.bq = sq; P.bw = w + 1; P.be = w + s.batch < size ? w + s.batch : size;
            P.mine += P.be - w;
            if (w + s.batch < size) {                  // claim the next batch early
                P.sq = sq; P.sw = atom_add_relaxed(q_head(s, sq), s.batch); P.spec = 1;
            }
            return q_pos(s, sq, w);
        }
        if (sq == P.q) {
            if (!s.steal || s.mode == MODE_IDENTITY) { P.q = -1; return -1; }
            // publish this agent's claims; if every slot of the launch is claimed
            // there is nothing left to steal (the returned value is consumed, so the
            // add is performed before this agent can reach its exit)
            const int32_t all = P.mine ? atom_add_relaxed(ws_claimed(s), P.mine) + P.mine
                                       : ld_relaxed(ws_claimed(s));
            P.mine = 0;
            if (all >= s.g.V) { P.q = -1; return -1; }
            *scan = 1;
            return -1;
        }
    }
}

// warp-parallel scan for a queue with unclaimed slots, nearest first from home.
// Each lane issues all its head loads (8 rounds of 32 queues) before any ballot,
// so a scan over up to 256 clusters costs one L2 round trip, not one per round.
__device__ __forceinline__ int32_t steal_scan(const Sched& s, int32_t home, int lane) {
    const int32_t M = s.g.M;
    for (int32_t base = 0; base < M; base += 256) {
        int32_t h[8], q[8];
#pragma unroll
        for (int r = 0; r < 8; ++r) {
            const int32_t k = base + r * 32 + lane;
            q[r] = -1;
            h[r] = 0;
            if (k < M) {
                int32_t qq = home + 1 + k;
                qq %= M;
                q[r] = qq;
                h[r] = ld_relaxed(ws_head(s) + qq);
            }
        }
#pragma unroll
        for (int r = 0; r < 8; ++r) {
            const bool avail = q[r] >= 0 && h[r] < cluster_size(s.g, q[r]);
            const uint32_t m = __ballot_sync(0xffffffffu, avail);
            if (m) return __shfl_sync(0xffffffffu, q[r], __ffs(m) - 1);
        }
    }
    return -1;
}

template <bool kStatic>
__device__ __forceinline__ int32_t producer_next(const Sched& s, Prod& P, int lane) {
    if constexpr (kStatic) {                               // CTA i owns cluster i: a local cursor
        int32_t v = -1;
        if (lane == 0 && P.q >= 0 && P.bw < cluster_size(s.g, P.q)) v = q_pos(s, P.q, P.bw++);
        return __shfl_sync(0xffffffffu, v, 0);
    }
    int32_t v = -1, scan = 0;
    if (lane == 0) v = lane0_next(s, P, &scan);
    scan = __shfl_sync(0xffffffffu, scan, 0);
    while (scan) {
        int32_t q = steal_scan(s, __shfl_sync(0xffffffffu, P.home, 0), lane);
        if (lane == 0) {
            if (q < 0) { P.q = -1; v = -1; scan = 0; }
            else { P.q = q; P.spec = 0; v = lane0_next(s, P, &scan); }
        }
        scan = __shfl_sync(0xffffffffu, scan, 0);
    }
    return __shfl_sync(0xffffffffu, v, 0);
}

// ---------------------------------------------------------------------------
// Body concept (see k_gemv.cuh / k_stencil.cuh / k_spmv.cuh):
//   kConsumers, kStageBytes, kDefaultStages, kDefaultBatch
//   produce(s, bx, by, stage, full, lane)  warp 0, all lanes: stage the task's
//                                       input and commit (stage_commit)
//   consume(bx, by, stage, ctid)        consumer threads ctid in [0, kConsumers)
//   finish(ctid)                        consumers, agent retiring: flush state
// ---------------------------------------------------------------------------
// ring buffer bytes per slot under STAGING_DIRECT: 128 unless the body's direct
// path stages for itself (it then uses its task's slot, which it owns until it
// releases the slot) and says how much with kDirectStageBytes
template <class B, class = void> struct DirectStageBytes { static constexpr int value = 128; };
template <class B> struct DirectStageBytes<B, decltype((void)B::kDirectStageBytes)> {
    static constexpr int value = B::kDirectStageBytes;
};
template <class B> constexpr int direct_stage_bytes() { return DirectStageBytes<B>::value; }

// Merged staging (kMerge = 2): a body may take two logical CTAs per ring slot
// when the scheduler pops them back to back and they are horizontal
// neighbours (same by, bx and bx+1) -- consecutive positions of a ROW or TILE
// cluster.  Their tiles share halo columns, so one wider copy stages both:
// the clustered order is what makes the pair co-located, and the shared
// halo is then reused from shared memory instead of being copied twice.
template <class B, class = void> struct MergeOf { static constexpr int value = 1; };
template <class B> struct MergeOf<B, decltype((void)B::kMerge)> { static constexpr int value = B::kMerge; };

struct RingShared {
    uint64_t full[MAX_STAGES];
    uint64_t empty[MAX_STAGES];
    int4 slot[MAX_STAGES];       // (v, lin, bx, by) decoded once by the scheduler warp
    int4 slot2[MAX_STAGES];      // merged slots: (v, lin) of the second CTA, and n
};

__device__ __forceinline__ uint8_t* ring_base(uint8_t* dyn) {
    const uint32_t a = smem_u32(dyn);
    return dyn + (((a + 127u) & ~127u) - a);
}

template <class Body, bool kStatic = false>
__device__ __forceinline__ void agent_loop(const Sched& s, Body& body) {
    extern __shared__ uint8_t dyn_smem[];
    __shared__ RingShared R;
    __shared__ int32_t s_active;
    uint8_t* ring = ring_base(dyn_smem);
    const int S = s.stages;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    constexpr int kConsumerWarps = Body::kConsumers / 32;
    if (threadIdx.x == 0) {
        for (int i = 0; i < S; ++i) { mbar_init(&R.full[i], 1); mbar_init(&R.empty[i], kConsumerWarps); }
        fence_mbar_init();
    }
    __syncthreads();
    if (warp == 0) {
        // ---- binding: dense SM rank from %smid, agent id by arrival
        Prod P{};
        int32_t active = 0;
        if constexpr (kStatic) {                               // binding by construction
            if (lane == 0) {
                P.q = (int32_t)blockIdx.x < s.g.M ? (int32_t)blockIdx.x : -1;
                P.bw = 0;
                s_active = active = 1;
            }
        } else if (lane == 0) {
            uint32_t sm = smid();
            int32_t rank = (int32_t)sm < s.smid_span ? s.rank_of_smid[sm] : -1;
            int32_t slot = (rank < 0 || rank >= s.g.M) ? s.g.M : rank;
            // agent id by arrival order (Listing 5 l.17-18) -- only needed to throttle
            int32_t a = s.throttle ? atom_add_relaxed(ws_agent_ctr(s) + slot, 1) : 0;
            if (rank >= s.g.M) rank = -1;                       // fewer clusters than SMs
            P.home = rank >= 0 ? rank : (int32_t)(blockIdx.x % (uint32_t)(s.g.M > 0 ? s.g.M : 1));
            P.q = (s.g.V > 0 && s.g.M > 0) ? P.home : -1;
            // throttling (Listing 5 l.20): agents past active_agents retire at once
            active = (a < s.active_agents) && (rank >= 0 || s.steal || s.mode == MODE_IDENTITY);
            if (!active) P.q = -1;
            if (s.mode == MODE_IDENTITY && active) P.q = 0;
            s_active = active;
        }
        // ---- producer ring (task t -> slot t % S, consumed by group t % G)
        int st = 0;
        uint32_t ph = 0;                                       // empty-barrier parity
        int32_t t = 0;
        int32_t pending = -1;                                  // popped but not yet staged (merge miss)
        __shared__ int32_t s_uwin[33];                         // USER-order window (lin_to_bxby_warp)
        if (lane == 0) s_uwin[0] = -64;
        __syncwarp();
        for (;; ++t) {
            if (t >= S) mbar_wait(&R.empty[st], ph ^ 1u);
            const int32_t v = pending >= 0 ? pending : producer_next<kStatic>(s, P, lane);
            pending = -1;
            if (v < 0) {
                if (lane == 0) R.slot[st] = make_int4(-1, 0, 0, 0);
                break;
            }
            int32_t lin, bx, by;
            lin_to_bxby_warp(s, s_uwin, v, lane, &lin, &bx, &by);
            if (lane == 0) R.slot[st] = make_int4(v, lin, bx, by);
            if constexpr (MergeOf<Body>::value > 1) {
                int n = 1;
                if (body.can_merge(s)) {
                    const int32_t v2 = producer_next<kStatic>(s, P, lane);
                    if (v2 >= 0) {
                        int32_t lin2, bx2, by2;
                        lin_to_bxby_warp(s, s_uwin, v2, lane, &lin2, &bx2, &by2);
                        if (by2 == by && bx2 == bx + 1) {
                            n = 2;
                            if (lane == 0) R.slot2[st] = make_int4(v2, lin2, n, 0);
                        } else if (by2 == by && bx2 == bx - 1) {       // popped right to left
                            n = 2;
                            if (lane == 0) {
                                R.slot[st] = make_int4(v2, lin2, bx2, by2);
                                R.slot2[st] = make_int4(v, lin, 2, 0);
                            }
                            bx = bx2;
                        } else {
                            pending = v2;                      // next slot starts with it
                        }
                    }
                }
                if (n == 1 && lane == 0) R.slot2[st] = make_int4(-1, 0, 1, 0);
                body.produce_n(s, bx, by, n, ring + (size_t)st * s.stage_bytes, &R.full[st], lane);
            } else {
                body.produce(s, bx, by, ring + (size_t)st * s.stage_bytes, &R.full[st], lane);
            }
            if (++st == S) { st = 0; ph ^= 1u; }
        }
        // one end marker per consumer group: slots t .. t+G-1
        for (int k = 0; k < Body::kGroups; ++k) {
            if (k > 0) {
                if (++st == S) { st = 0; ph ^= 1u; }
                if (t + k >= S) mbar_wait(&R.empty[st], ph ^ 1u);
                if (lane == 0) R.slot[st] = make_int4(-1, 0, 0, 0);
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&R.full[st]);
        }
        // ---- the last agent out resets the workspace for the next launch.  Every
        // other agent's producer has consumed the results of all its atomics
        // (including any speculative claim) before arriving here.
        int32_t last = 0;
        if (lane == 0 && !kStatic) {                           // the static backend has no workspace
            const int32_t total = (int32_t)(gridDim.x * gridDim.y * gridDim.z);
            last = atom_add_relaxed(ws_done(s), 1) == total - 1;
        }
        if (__shfl_sync(0xffffffffu, last, 0)) {
            const int32_t n = 2 * s.g.M + 4;
            for (int32_t k = lane; k < n; k += 32) s.ws[k] = 0;
        }
    } else {
        const int grp = (threadIdx.x - PRODUCER_THREADS) / Body::kConsumers;
        const int ctid = (threadIdx.x - PRODUCER_THREADS) % Body::kConsumers;
        int st = grp;                                          // group g takes tasks g, g+G, ...
        uint32_t ph = 0;                                       // full-barrier parity (G <= S)
        for (;;) {
            mbar_wait(&R.full[st], ph);
            // lane 0 reads the slot descriptor and broadcasts it: the lane that
            // later releases the slot (arrive on empty) is the only one that
            // read it, so the producer's next write is ordered after every read
            // by that arrive alone (compute-sanitizer racecheck is clean)
            int4 sl = make_int4(0, 0, 0, 0), s2 = make_int4(0, 0, 1, 0);
            if (lane == 0) {
                sl = R.slot[st];
                if constexpr (MergeOf<Body>::value > 1) s2 = R.slot2[st];
            }
            sl.x = __shfl_sync(0xffffffffu, sl.x, 0);
            sl.y = __shfl_sync(0xffffffffu, sl.y, 0);
            sl.z = __shfl_sync(0xffffffffu, sl.z, 0);
            sl.w = __shfl_sync(0xffffffffu, sl.w, 0);
            if (sl.x < 0) break;
            if constexpr (MergeOf<Body>::value > 1) {
                s2.x = __shfl_sync(0xffffffffu, s2.x, 0);
                s2.y = __shfl_sync(0xffffffffu, s2.y, 0);
                s2.z = __shfl_sync(0xffffffffu, s2.z, 0);
                body.consume_n(s, sl.z, sl.w, s2.z, ring + (size_t)st * s.stage_bytes, ctid);
                if (ctid == 0) {
                    record(s, sl.x, sl.y);
                    if (s2.z > 1) record(s, s2.x, s2.y);
                }
            } else {
                body.consume(s, sl.z, sl.w, ring + (size_t)st * s.stage_bytes, ctid);
                if (ctid == 0) record(s, sl.x, sl.y);
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&R.empty[st]);
            st += Body::kGroups;
            if (st >= S) { st -= S; ph ^= 1u; }
        }
        if (s_active) body.finish(ctid);
    }
}

// One-shot CTA (default hardware order, or redirection): the same producer /
// consumer split with a single stage and a single task.
template <class Body>
__device__ __forceinline__ void one_shot(const Sched& s, Body& body, int32_t v, int32_t lin, int32_t bx, int32_t by) {
    extern __shared__ uint8_t dyn_smem[];
    __shared__ uint64_t full;
    uint8_t* ring = ring_base(dyn_smem);
    if (threadIdx.x == 0) { mbar_init(&full, 1); fence_mbar_init(); }
    __syncthreads();
    if (threadIdx.x < PRODUCER_THREADS) {
        body.produce(s, bx, by, ring, &full, threadIdx.x);
    } else {
        const int ctid = threadIdx.x - PRODUCER_THREADS;
        mbar_wait(&full, 0);
        body.consume(s, bx, by, ring, ctid);
        if (ctid == 0) {
            if (s.census) atomicAdd(s.census + lin, 1u);
            if (s.exec_sm) s.exec_sm[lin] = (int32_t)smid();
            if (s.map && v >= 0) s.map[v] = lin;
        }
        body.finish(ctid);
    }
}

// ---- kernels: one per (body, backend) ------------------------------------
template <class Body>
__global__ void __launch_bounds__(Body::kGroups * Body::kConsumers + PRODUCER_THREADS, Body::kMinAgents)
k_agent(const __grid_constant__ Sched s, const __grid_constant__ typename Body::Params p) {
    Body body(p);
    body.l2h = s.l2_hint;        // L2 hints ride with clustering (CLU+BPS); one-shot kernels compile them out
    agent_loop(s, body);
}

// static binding (CC_BACKEND_AGENT_STATIC): grid = M, CTA i runs cluster i
template <class Body>
__global__ void __launch_bounds__(Body::kGroups * Body::kConsumers + PRODUCER_THREADS, Body::kMinAgents)
k_static(const __grid_constant__ Sched s, const __grid_constant__ typename Body::Params p) {
    Body body(p);
    body.l2h = s.l2_hint;
    agent_loop<Body, true>(s, body);
}

template <class Body>
__global__ void __launch_bounds__(Body::kConsumers + PRODUCER_THREADS) k_default(const __grid_constant__ Sched s,
                                                                             const __grid_constant__ typename Body::Params p) {
    Body body(p);
    const int32_t bx = blockIdx.x, by = blockIdx.y;
    one_shot(s, body, -1, by * s.g.gx + bx, bx, by);
}

// Redirection-based clustering (Listing 4, Fig. 9): same number of CTAs as O;
// CTA u runs v = rd_redirect(u).
template <class Body>
__global__ void __launch_bounds__(Body::kConsumers + PRODUCER_THREADS) k_redirect(const __grid_constant__ Sched s,
                                                                              const __grid_constant__ typename Body::Params p) {
    Body body(p);
    const int32_t v = rd_redirect(s.g, (int32_t)blockIdx.x);
    int32_t lin, bx, by;
    lin_to_bxby(s, v, &lin, &bx, &by);
    one_shot(s, body, v, lin, bx, by);
}

}  // namespace cc
