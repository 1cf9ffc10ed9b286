// k_jwave.cuh -- K fused Jacobi sweeps as column-strip wavefronts carried from
// one logical CTA to the next (CC_K_JACOBI5_WAVE, reading R34).
//
// Clustering puts logical CTAs that share data on one SM (§4.2,
// P:1793); agent-based clustering runs a cluster's CTAs back to back on the
// SM's agents (Listing 5).  Here the shared data between vertically
// adjacent tiles of K fused sweeps is the 2K-row band where their light cones
// overlap; when an agent's next logical CTA is the tile directly below its
// last one (consecutive positions of a COL (X-P) cluster), it keeps
// that band -- the last two rows of every intermediate sweep -- in registers
// and streams on, so the band is neither re-read nor recomputed.  Any other
// successor (identity / ROW order, hardware order) starts afresh: 2K rows
// re-read and re-swept.
//
// Agent = one warp.  Logical CTA (bx, by) = output rows [64 by, 64 by + 64) x
// columns [WS bx, WS bx + WS), WS = 128 - 8 HL; the warp streams the strip's
// 128 loaded columns (4 per lane, 4 HL halo columns each side) row by row
// through a per-warp cp.async ring of JW_DEPTH rows.  Ingesting input row i
// yields sweep 1 on row i-1, sweep 2 on row i-2, ..., sweep K on row i-K
// (stored): sweep l+1 on row j needs sweep l on rows j-1, j, j+1, which are
// three registers per lane and level (a rotation unrolled over the ingest
// count mod 3) and the value just produced; the horizontal
// neighbours are the adjacent lanes' edge columns (two shuffles per sweep).
// A lane's garbage neighbour at the strip edge reaches one column further per
// sweep, so the 4 HL >= K edge columns absorb it.  Each point is computed
// with jacobi_core4's single-sweep expression (PolyBench order, R14) and the
// boundary rows / columns are copied, so K fused sweeps are bit-identical to
// K single sweeps.
//
// The runtime around the body is generic (k_strip<Body, KIND>): one-shot
// warps in hardware order, or persistent workers -- one CTA per SM, its last
// warp a scheduler that binds to the SM's cluster, claims chunks of the
// cluster queue (then single tiles, then steals) and posts each worker's next
// logical CTAs into a shared-memory mailbox, so the workers' row loop carries
// no scheduler code next to the sweep registers.
#pragma once
#include <stdint.h>
#include <type_traits>
#include "cc_runtime.cuh"
#include "k_stencil.cuh"

namespace cc {

constexpr int JW_ROWS = 64;     // default output rows per logical CTA (cc_jacobi5_args.tile_rows = 0)
constexpr int JW_WARPS = 8;     // worker warps per CTA of the one-shot kernel
constexpr int JW_DEPTH = 8;     // rows in flight per warp (cp.async ring)
constexpr int JW_BATCH = 0;     // default claim size: 0 = chunked claims (jw_claim)
#ifndef JW_TAIL
#define JW_TAIL 4               // chunked claims: the last 1/JW_TAIL of a queue goes tile by tile
#endif
enum : int { JW_DYNAMIC = 0, JW_STATIC = 1, JW_ONESHOT = 2 };

__host__ __device__ constexpr int jw_halo_chunks(int K) { return K <= 4 ? 1 : 2; }
__host__ __device__ constexpr int jw_strip_cols(int hl) { return 128 - 8 * hl; }

struct JWaveParams { const float* a; float* b; int64_t ld; int32_t rows, cols; int32_t trows; };

// one vertical run of logical CTAs of strip bx: output rows [e0, e1), input
// rows [e0 - K, e1 + K) streamed
struct JwRun { int32_t bx, e0, e1; };

__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
// wait until at most n of this thread's cp.async groups are pending
__device__ __forceinline__ void cp_async_wait_dyn(int n) {
    switch (n) {
    case 0: asm volatile("cp.async.wait_group 0;" ::: "memory"); break;
    case 1: asm volatile("cp.async.wait_group 1;" ::: "memory"); break;
    case 2: asm volatile("cp.async.wait_group 2;" ::: "memory"); break;
    case 3: asm volatile("cp.async.wait_group 3;" ::: "memory"); break;
    case 4: asm volatile("cp.async.wait_group 4;" ::: "memory"); break;
    case 5: asm volatile("cp.async.wait_group 5;" ::: "memory"); break;
    default: asm volatile("cp.async.wait_group 6;" ::: "memory"); break;
    }
}
static_assert(JW_DEPTH - 2 <= 6, "cp_async_wait_dyn covers JW_DEPTH - 2 pending groups");

// Ingest input row i (x = this lane's 4 columns): advance every sweep level
// by one row and return sweep K on row i - K.  S[l][*] holds sweep l's last
// two rows in a three-slot rotation: at phase PH (= ingest count mod 3, a
// template parameter, so the rotation costs no moves) row j-1 is in slot
// PH+1, row j in slot PH+2, and row j+1 (produced now) replaces row j-1 in
// slot PH.  SLOW: some row of i-K .. i-1 is a boundary row (0 or rows - 1,
// copied) or the strip holds a boundary column (keep: this lane's global
// boundary columns, bit e = column 4 lane + e); otherwise no selects at all.
template <int K, int PH, bool SLOW>
__device__ __forceinline__ float4 jw_ingest(float4 (&S)[K][3], float4 x, int32_t i, int32_t rows, uint32_t keep) {
    float4 nw = x;
#pragma unroll
    for (int l = 0; l < K; ++l) {
        const float4 up = S[l][(PH + 1) % 3];
        const float4 c = S[l][(PH + 2) % 3];
        const float lw = __shfl_up_sync(0xffffffffu, c.w, 1);
        const float re = __shfl_down_sync(0xffffffffu, c.x, 1);
        float4 o = jacobi_core4(c, up, nw, lw, re);
        if (SLOW) {
            const int32_t j = i - l - 1;                  // row of sweep l + 1 produced now (warp-uniform)
            const bool bd = j == 0 || j == rows - 1;
            if (bd || (keep & 1u)) o.x = c.x;
            if (bd || (keep & 2u)) o.y = c.y;
            if (bd || (keep & 4u)) o.z = c.z;
            if (bd || (keep & 8u)) o.w = c.w;
        }
        S[l][PH] = nw;
        nw = o;
    }
    return nw;
}

// Scheduler state of one warp agent, in shared memory between pops (lane 0
// owns it; the registers belong to the sweep levels the hot loop keeps live).
struct JwSched {
    int32_t q;        // queue being drained (-1: none left); static: the agent's cluster
    int32_t home;     // home queue (steal scan start)
    int32_t bq, bw, be;   // current run: slots [bw, be) of queue bq
    int32_t cdone;    // no chunk of queue q left to claim
};

// Chunked queues (s.batch == 0, the default).  The first 3/4 of a queue's
// slots are cut into A contiguous chunks, A = the agents sharing the queue;
// an agent claims a whole chunk (one counter per queue) and runs it as one
// vertical run -- continuation all the way down.  The last quarter is popped
// one slot at a time, by the queue's agents and then by thieves, so agents
// that finish early absorb the imbalance between SMs (a persistent agent
// cannot hand work back to the hardware scheduler).  s.batch > 0: plain
// claims of s.batch slots.
__device__ __forceinline__ int32_t jw_agents(const Sched& s) {
    return s.mode == MODE_IDENTITY ? s.active_agents * s.g.M : s.active_agents;
}
__device__ __forceinline__ int32_t jw_split(int32_t n) { return n - n / JW_TAIL; }
__device__ __forceinline__ int32_t* jw_chunk_ctr(const Sched& s, int32_t q) {
    return ws_chunk(s) + (s.mode == MODE_IDENTITY ? 0 : q);
}

// Warp-parallel scan for a queue with unclaimed slots, nearest first from
// home; one 32-queue round at a time (few registers: steals happen once per
// agent, at its end).  -1: every queue is drained.
__device__ __forceinline__ int32_t jw_steal_scan(const Sched& s, int32_t home, int lane) {
    const int32_t M = s.g.M;
    const int32_t A = jw_agents(s);
    for (int32_t base = 0; base < M; base += 32) {
        const int32_t k = base + lane;
        int32_t q = -1;
        bool avail = false;
        if (k < M) {
            q = home + 1 + k;
            if (q >= M) q -= M;
            const int32_t n = cluster_size(s.g, q);
            if (s.batch > 0) avail = ld_relaxed(ws_head(s) + q) < n;
            else avail = ld_relaxed(ws_chunk(s) + q) < A || ld_relaxed(ws_head(s) + q) < n - jw_split(n);
        }
        const uint32_t m = __ballot_sync(0xffffffffu, avail);
        if (m) return __shfl_sync(0xffffffffu, q, __ffs(m) - 1);
    }
    return -1;
}

// lane 0: one claim on queue P.q; returns a position (and sets up the run in
// P) or -1 when the queue has nothing left
__device__ __forceinline__ int32_t jw_claim(const Sched& s, JwSched& P) {
    const int32_t n = q_size(s, P.q);
    if (s.batch > 0) {
        const int32_t w = atom_add_relaxed(q_head(s, P.q), s.batch);
        if (w >= n) return -1;
        P.bq = P.q; P.bw = w + 1; P.be = w + s.batch < n ? w + s.batch : n;
        return q_pos(s, P.q, w);
    }
    const int32_t split = jw_split(n), A = jw_agents(s);
    while (!P.cdone) {
        const int32_t c = atom_add_relaxed(jw_chunk_ctr(s, P.q), 1);
        if (c >= A) { P.cdone = 1; break; }
        const int32_t lo = (int32_t)((int64_t)c * split / A), hi = (int32_t)((int64_t)(c + 1) * split / A);
        if (lo < hi) {
            P.bq = P.q; P.bw = lo + 1; P.be = hi;
            return q_pos(s, P.q, lo);
        }
    }
    const int32_t w = atom_add_relaxed(q_head(s, P.q), 1);
    return split + w < n ? q_pos(s, P.q, split + w) : -1;
}

// Next order position of a warp agent (all lanes; -1: done).  STATIC: the
// agent's own cluster front to back (Eq. 7 order), no atomics.  Otherwise
// claims on the cluster queue (identity: the one global row-major queue),
// then steals (R9/R10), as the CTA agents' scheduler.
template <int KIND>
__device__ __forceinline__ int32_t jw_next(const Sched& s, JwSched& P, int lane) {
    if constexpr (KIND == JW_STATIC) {
        int32_t v = -1;
        if (P.q >= 0 && P.bw < cluster_size(s.g, P.q)) v = cluster_start(s.g, P.q) + P.bw++;
        return v;                                           // P is warp-uniform here: every lane steps it
    } else {
        int32_t v = -1, scan = 0;
        for (;;) {
            if (lane == 0) {
                scan = 0;
                if (P.bw < P.be) {
                    v = q_pos(s, P.bq, P.bw++);
                } else if (P.q >= 0) {
                    v = jw_claim(s, P);
                    if (v < 0) {
                        if (s.steal && s.mode != MODE_IDENTITY) scan = 1;
                        else P.q = -1;
                    }
                }
            }
            if (!__shfl_sync(0xffffffffu, scan, 0)) break;
            const int32_t q = jw_steal_scan(s, __shfl_sync(0xffffffffu, P.home, 0), lane);
            if (lane == 0) { P.q = q; P.cdone = 0; }
        }
        return __shfl_sync(0xffffffffu, v, 0);
    }
}

// Task mailboxes (persistent kinds): the CTA's last warp is a scheduler that
// pops logical CTAs for the worker warps and posts them, JW_MB ahead, into
// one small ring per worker; a worker's pop is a shared-memory read.  Workers
// thus carry none of the scheduler's code (atomics, steal scan, USER window,
// census) -- a pop inline or as a call in the row loop cost them registers
// (spills next to the sweep levels: measured 15-25 % slower, ncu jw3).
constexpr int JW_MB = 4;
struct JwSlot { int32_t bx, by, seq, pad; };
__device__ __forceinline__ int32_t ld_acquire_cta(const int32_t* p) {
    int32_t v;
    asm volatile("ld.acquire.cta.shared::cta.b32 %0, [%1];" : "=r"(v) : "r"(smem_u32(p)) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_cta(int32_t* p, int32_t v) {
    asm volatile("st.release.cta.shared::cta.b32 [%0], %1;" :: "r"(smem_u32(p)), "r"(v) : "memory");
}

// ---------------------------------------------------------------------------
// Strip bodies.  A body says what one ingested input row does to a warp's
// registers: kVec float4 per lane (a strip is 128 kVec loaded columns),
// kHaloLanes lanes at each strip edge that load but do not store (the output
// strip is WS = (32 - 2 kHaloLanes) 4 kVec columns), kLag (ingesting row i
// yields output row i - kLag, so a fresh run starts kLag rows above its first
// output row), kPhases (the ingest count modulo which the body rotates its
// registers, a template parameter of ingest()).
// ---------------------------------------------------------------------------

// Jacobi, K fused sweeps (R34)
template <int K, int HL>
struct JwJacobi {
    static constexpr int kVec = 1, kHaloLanes = HL, kLag = K, kPhases = 3;
    static constexpr int kWorkers = K <= 3 ? 24 : K == 4 ? 20 : 15;   // persistent kinds, one CTA per SM
    static constexpr int kOneshotBlocks = K <= 4 ? 3 : 2;
    static_assert(K >= 1 && 4 * HL >= K, "the strip's halo columns must cover K sweeps");
    using Params = JWaveParams;
    float4 S[K][3];
    uint32_t keep;          // this lane's global boundary columns (bit e = column gcol + e)
    bool edge;              // the strip holds a boundary column
    __device__ __forceinline__ void init(const Params&) {
#pragma unroll
        for (int l = 0; l < K; ++l)
#pragma unroll
            for (int m = 0; m < 3; ++m) S[l][m] = make_float4(0.f, 0.f, 0.f, 0.f);
    }
    // per strip: returns this lane's store kind (0 none, 1 full float4s, 2 masked ragged edge)
    __device__ __forceinline__ int32_t set_strip(int32_t gcol, int lane, const Params& p) {
        const int32_t cols = p.cols;
        keep = 0;
#pragma unroll
        for (int e = 0; e < 4; ++e)
            if (gcol + e == 0 || gcol + e == cols - 1) keep |= 1u << e;
        edge = __any_sync(0xffffffffu, keep != 0);
        return (lane < HL || lane >= 32 - HL || gcol >= cols) ? 0 : (gcol + 3 < cols ? 1 : 2);
    }
    template <int PH>
    __device__ __forceinline__ void ingest(const float4 (&x)[1], int32_t i, float4 (&o)[1], const Params& p) {
        const int32_t rows = p.rows;
        const bool slow = edge || (uint32_t)(i - 1) < (uint32_t)K || (uint32_t)(i - rows) < (uint32_t)K;
        o[0] = slow ? jw_ingest<K, PH, true>(S, x[0], i, rows, keep) : jw_ingest<K, PH, false>(S, x[0], i, rows, keep);
    }
};

// Worker warps per CTA.  One-shot: JW_WARPS per CTA, B::kOneshotBlocks CTAs
// per SM.  Persistent kinds: ONE CTA per SM, B::kWorkers workers plus one
// scheduler warp, sized so that a thread keeps the registers the body needs
// (65536 / threads: 24 + 1 warps -> 80, 20 + 1 -> 96, 15 + 1 -> 128); more
// workers and ptxas moves the body's registers to local memory (measured:
// 15-25 % slower).
template <class B> __host__ __device__ constexpr int jw_workers(int kind) {
    return kind == JW_ONESHOT ? JW_WARPS : B::kWorkers;
}
template <class B> __host__ __device__ constexpr int jw_threads(int kind) {
    return (jw_workers<B>(kind) + (kind == JW_ONESHOT ? 0 : 1)) * 32;
}
// dynamic shared memory: the workers' cp.async rings
template <class B> __host__ __device__ constexpr int jw_smem(int kind) {
    return jw_workers<B>(kind) * JW_DEPTH * 32 * 16 * B::kVec;
}
template <class B> __host__ __device__ constexpr int jw_ws() { return (32 - 2 * B::kHaloLanes) * 4 * B::kVec; }

template <class B, int KIND>
__global__ void __launch_bounds__(jw_threads<B>(KIND), (KIND == JW_ONESHOT ? B::kOneshotBlocks : 1))
k_strip(const __grid_constant__ Sched s, const __grid_constant__ typename B::Params p) {
    constexpr int NW = jw_workers<B>(KIND);                              // worker warps
    constexpr int V = B::kVec, LAG = B::kLag;
    constexpr int WS = jw_ws<B>();
    constexpr int HC = 4 * V * B::kHaloLanes;                            // halo columns per side
    static_assert(NW < 32, "live-worker mask");
    extern __shared__ __align__(16) float4 jw_dyn[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int32_t rows = p.rows, cols = p.cols;
    const int64_t ld = p.ld;
    __shared__ JwSlot mb[NW][JW_MB];
    __shared__ int32_t mcons[NW];

    if constexpr (KIND != JW_ONESHOT) {
        if (threadIdx.x < NW * JW_MB) mb[threadIdx.x / JW_MB][threadIdx.x % JW_MB].seq = 0;
        if (threadIdx.x < NW) mcons[threadIdx.x] = 0;
        __syncthreads();
        if (warp == NW) {
            // ================= scheduler warp =================
            __shared__ JwSched sP[NW];
            __shared__ int32_t sprod[NW];
            __shared__ int32_t uwin[33];
            if (lane == 0) {
                uwin[0] = -64;
                const uint32_t sm = smid();
                int32_t rank = (int32_t)sm < s.smid_span ? s.rank_of_smid[sm] : -1;
                const int32_t slot = (rank < 0 || rank >= s.g.M) ? s.g.M : rank;
                if (rank >= s.g.M) rank = -1;
                for (int w = 0; w < NW; ++w) {
                    JwSched P{};
                    P.bw = P.be = 0;
                    P.cdone = 0;
                    const int32_t agent = (int32_t)blockIdx.x * NW + w;
                    if constexpr (KIND == JW_STATIC) {
                        P.q = agent < s.g.M ? agent : -1;                // agent i runs cluster i
                    } else {
                        // binding: the SM's cluster; agent id by
                        // arrival order (Listing 5 l.17-18), only needed to throttle
                        const int32_t a = s.throttle ? atom_add_relaxed(ws_agent_ctr(s) + slot, 1) : 0;
                        P.home = rank >= 0 ? rank : agent % (s.g.M > 0 ? s.g.M : 1);
                        P.q = (s.g.V > 0 && s.g.M > 0) ? P.home : -1;
                        const bool active = (a < s.active_agents) && (rank >= 0 || s.steal || s.mode == MODE_IDENTITY);
                        if (!active) P.q = -1;
                        if (s.mode == MODE_IDENTITY && active) P.q = 0;
                    }
                    sP[w] = P;
                    sprod[w] = 0;
                }
            }
            __syncwarp();
            uint32_t live = (1u << NW) - 1u;
            while (live) {
                bool posted = false;
                for (int w = 0; w < NW; ++w) {
                    if (!((live >> w) & 1u)) continue;
                    const int32_t k = sprod[w];
                    if (k - ld_acquire_cta(&mcons[w]) >= JW_MB) continue;
                    JwSched P = sP[w];
                    const int32_t v = jw_next<KIND>(s, P, lane);
                    int32_t lin = 0, bx = -1, by = 0;
                    if (v >= 0) {
                        lin_to_bxby_warp(s, uwin, v, lane, &lin, &bx, &by);
                        if (lane == 0) record(s, v, lin);
                    } else {
                        live &= ~(1u << w);
                    }
                    __syncwarp();
                    if (lane == 0) {
                        sP[w] = P;
                        sprod[w] = k + 1;
                        JwSlot& e = mb[w][k % JW_MB];
                        e.bx = bx;
                        e.by = by;
                        st_release_cta(&e.seq, k + 1);
                    }
                    __syncwarp();
                    posted = true;
                }
                if (!posted) __nanosleep(256);
            }
            // ---- the last scheduler out resets the workspace for the next launch
            if constexpr (KIND == JW_DYNAMIC) {
                int32_t last = 0;
                if (lane == 0) last = atom_add_relaxed(ws_done(s), 1) == (int32_t)gridDim.x - 1;
                if (__shfl_sync(0xffffffffu, last, 0)) {
                    const int32_t n = 3 * s.g.M + 4;                    // ws_ints: incl. the chunk counters
                    for (int32_t k = lane; k < n; k += 32) s.ws[k] = 0;
                }
            }
            return;
        }
    }

    // ================= worker warps =================
    int32_t oneshot = -1, taken = 0;
    if constexpr (KIND == JW_ONESHOT) {
        const int32_t gw = (int32_t)blockIdx.x * NW + warp;
        oneshot = gw < s.g.V ? gw : -1;                       // hardware order: warp = logical CTA lin
    }
    // next logical CTA of this agent (warp-uniform)
    auto pop = [&](JwRun& r) -> bool {
        int32_t bx, by;
        if constexpr (KIND == JW_ONESHOT) {
            if (oneshot < 0) return false;
            const int32_t lin = oneshot;
            oneshot = -1;
            by = lin / s.g.gx; bx = lin - by * s.g.gx;
            if (lane == 0) {
                if (s.census) atomicAdd(s.census + lin, 1u);
                if (s.exec_sm) s.exec_sm[lin] = (int32_t)smid();
            }
        } else {
            JwSlot& e = mb[warp][taken % JW_MB];
            while (ld_acquire_cta(&e.seq) != taken + 1) __nanosleep(32);
            bx = *(volatile int32_t*)&e.bx;
            by = *(volatile int32_t*)&e.by;
            ++taken;
            __syncwarp();
            if (lane == 0) st_release_cta(&mcons[warp], taken);
            if (bx < 0) return false;
        }
        r.bx = bx;
        r.e0 = by * p.trows;                                  // logical CTA height (parameter bank)
        r.e1 = r.e0 + p.trows < rows ? r.e0 + p.trows : rows;
        return true;
    };

    // Run bookkeeping touched only when a run ends or the prefetch cursor
    // leaves one lives in shared memory; the registers hold the body's state
    // and the per-row cursors.
    struct JwWarp { JwRun nxt; int32_t cur_bx, cur_e1, has_nxt, more, pf_in_nxt, pf_done; };
    __shared__ JwWarp sW[NW];
    JwWarp& W = sW[warp];
    auto wset = [&](int32_t& f, int32_t v) { __syncwarp(); if (lane == 0) f = v; __syncwarp(); };
    JwRun first;
    if (pop(first)) {
        if (lane == 0) { W.cur_bx = first.bx; W.cur_e1 = first.e1; W.has_nxt = 0; W.more = 1; W.pf_in_nxt = 0; W.pf_done = 0; }
        __syncwarp();
        // this lane's ring entries as a 32-bit shared address ([slot][lane][v], slot stride 32 V float4):
        // one register, no generic-to-shared conversion per row
        const uint32_t my = smem_u32(jw_dyn) + (uint32_t)(((warp * JW_DEPTH * 32) + lane) * V * 16);
        // ---- prefetch cursor: rows [pf_row, pf_end) from pf_ptr on; pf_ok: this
        // lane's float4 chunks inside the image (bit v)
        int32_t pf_row = 0, pf_end = 0;
        uint32_t pf_ok = 0;
        const float* pf_ptr = p.a;
        auto pf_start = [&](const JwRun& r) {
            const int32_t gcol = r.bx * WS - HC + 4 * V * lane;
            pf_row = r.e0 - LAG;
            pf_end = r.e1 + LAG;
            uint32_t ok = 0;
#pragma unroll
            for (int v = 0; v < V; ++v)
                if (gcol + 4 * v >= 0 && gcol + 4 * v < cols) ok |= 1u << v;
            if constexpr (V > 1) pf_ok = ok;
            // one float4 per lane: a null cursor says "outside" (no mask register)
            pf_ptr = ok ? p.a + (int64_t)pf_row * ld + gcol : (V > 1 ? p.a : nullptr);
        };
        pf_start(first);
        int32_t n_iss = 0, n_use = 0;            // rows issued / consumed (one cp.async group each)
        B body;
        body.init(p);
        // ---- consumer cursor: ingest row i < i_end of the current run, store
        // row i - LAG (through st_ptr) once i >= st_from
        int32_t i = 0, i_end = 0, st_from = 0, st_kind = 0;
        float* st_ptr = p.b;
        auto set_strip = [&](const JwRun& r) {
            i = r.e0 - LAG;
            i_end = r.e1 + LAG;
            st_from = r.e0 + LAG;
            const int32_t gcol = r.bx * WS - HC + 4 * V * lane;
            st_kind = body.set_strip(gcol, lane, p);
            st_ptr = p.b + (int64_t)(i - LAG) * ld + (st_kind ? gcol : 0);
        };
        set_strip(first);
        // the prefetch cursor ran off its run: extend the current run when the
        // agent's next logical CTA continues it (same strip, directly below),
        // else move on to the next run (rare: once per logical CTA at most)
        auto refill = [&]() -> bool {
            if (W.pf_done || W.pf_in_nxt) return false;
            if (!W.has_nxt && W.more) {
                JwRun r;
                if (pop(r)) {
                    if (r.bx == W.cur_bx && r.e0 == W.cur_e1) {       // continuation
                        const int32_t d = r.e1 - W.cur_e1;
                        pf_end += d;
                        i_end += d;
                        wset(W.cur_e1, r.e1);
                        return true;
                    }
                    __syncwarp();
                    if (lane == 0) { W.nxt = r; W.has_nxt = 1; }
                    __syncwarp();
                } else {
                    wset(W.more, 0);
                }
            }
            if (W.has_nxt) { wset(W.pf_in_nxt, 1); pf_start(W.nxt); return true; }
            wset(W.pf_done, 1);
            return false;
        };
        auto issue_one = [&]() -> bool {
            if (pf_row >= pf_end && !refill()) return false;
            const bool row_in = (uint32_t)pf_row < (uint32_t)rows;
            const uint32_t dst = my + (uint32_t)(n_iss % JW_DEPTH) * (32 * V * 16);
#pragma unroll
            for (int v = 0; v < V; ++v) {
                const bool in = row_in && (V > 1 ? ((pf_ok >> v) & 1u) != 0 : pf_ptr != nullptr);
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;"
                             :: "r"(dst + 16 * v), "l"(in ? pf_ptr + 4 * v : p.a), "r"(in ? 16u : 0u) : "memory");
            }
            cp_async_commit();
            if (V > 1 ? pf_ok != 0 : pf_ptr != nullptr) pf_ptr += ld;
            ++pf_row;
            ++n_iss;
            return true;
        };
        while (n_iss < JW_DEPTH - 1 && issue_one()) {}

        // one ingested row; the phase (ingest count mod kPhases) picks the body's register rotation
        auto step = [&](auto phase) -> bool {
            constexpr int PH = decltype(phase)::value;
            if (i >= i_end) {
                if (!W.has_nxt) return false;
                const JwRun r = W.nxt;                             // a fresh run: the body restarts
                __syncwarp();
                if (lane == 0) { W.has_nxt = 0; W.pf_in_nxt = 0; W.cur_bx = r.bx; W.cur_e1 = r.e1; }
                __syncwarp();
                set_strip(r);
            }
            const int ahead = n_iss - n_use - 1;                   // groups issued after row i's
            if (ahead >= JW_DEPTH - 2) asm volatile("cp.async.wait_group %0;" :: "n"(JW_DEPTH - 2) : "memory");
            else cp_async_wait_dyn(ahead);
            float4 x[V], o[V];
            const uint32_t src = my + (uint32_t)(n_use % JW_DEPTH) * (32 * V * 16);
#pragma unroll
            for (int v = 0; v < V; ++v)
                asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                             : "=f"(x[v].x), "=f"(x[v].y), "=f"(x[v].z), "=f"(x[v].w) : "r"(src + 16 * v) : "memory");
            ++n_use;
            if (n_iss - n_use < JW_DEPTH - 1) issue_one();
            body.template ingest<PH>(x, i, o, p);
            if (st_kind && i >= st_from) {
                if (st_kind == 2) {                                // ragged right edge (rare): column from smem
                    const int32_t gcol = W.cur_bx * WS - HC + 4 * V * lane;
#pragma unroll
                    for (int v = 0; v < V; ++v)
                        if (gcol + 4 * v < cols) store4_masked(st_ptr + 4 * v, o[v], gcol + 4 * v, cols);
                } else {
#pragma unroll
                    for (int v = 0; v < V; ++v) *reinterpret_cast<float4*>(st_ptr + 4 * v) = o[v];
                }
            }
            st_ptr += ld;
            ++i;
            return true;
        };
        constexpr int NP = B::kPhases;
        static_assert(NP >= 1 && NP <= 7, "phases");
        for (;;) {
            if (!step(std::integral_constant<int, 0>{})) break;
            if constexpr (NP > 1) if (!step(std::integral_constant<int, 1 % NP>{})) break;
            if constexpr (NP > 2) if (!step(std::integral_constant<int, 2 % NP>{})) break;
            if constexpr (NP > 3) if (!step(std::integral_constant<int, 3 % NP>{})) break;
            if constexpr (NP > 4) if (!step(std::integral_constant<int, 4 % NP>{})) break;
            if constexpr (NP > 5) if (!step(std::integral_constant<int, 5 % NP>{})) break;
            if constexpr (NP > 6) if (!step(std::integral_constant<int, 6 % NP>{})) break;
        }
        asm volatile("cp.async.wait_all;" ::: "memory");
    }
}

}  // namespace cc
