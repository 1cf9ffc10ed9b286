// cc_runtime.cuh -- the agent runtime (binding + task loop) for sm_100a.
//
// PAPER.md §4.2.3 Step 3 "Binding", §4.2.4(2) agent-based
// clustering (Fig. 8(D), Listing 5) and §4.3(I) CTA throttling
// (P:2183).  B200-first differences from Listing 5:
//   * cluster i binds to the SM of dense rank i from a probe-built table, not to
//     raw %smid (virtual, possibly sparse; reading R7);
//   * agents pop slots from a per-cluster queue with relaxed atomics instead of
//     a static stride v += ACTIVE_AGENTS, and steal from other clusters when
//     their own is empty, so coverage is exactly-once even if the hardware
//     places fewer agents on an SM than expected (reading R10);
//   * the pop for the next task is issued before the current body runs and only
//     consumed after it, hiding the L2 atomic round trip;
//   * no gpu-scope fence or acquire anywhere in the loop: on sm_100a those emit
//     CCTL.IVALL, which would wipe the very L1 contents clustering tries to keep;
//   * the workspace resets itself: the last agent to leave zeroes the counters,
//     so a launch is one kernel (no memset node).
#pragma once
#include <stdint.h>
#include <cuda_runtime.h>
#include "cc_index.cuh"

namespace cc {

enum : int32_t { MODE_AGENT = 0, MODE_IDENTITY = 1 };

// Everything a task loop needs, passed by value as a kernel parameter.
struct Sched {
    Grid g;
    const int32_t* user;          // USER order table: v -> lin (device)
    const int32_t* rank_of_smid;  // %smid -> dense SM rank or -1 (device)
    int32_t smid_span;
    int32_t* ws;                  // workspace: agent_ctr[M+1] | head[M] | gq | done
    int32_t mode;                 // MODE_AGENT / MODE_IDENTITY
    int32_t active_agents;
    int32_t steal;
    int32_t prefetch;
    uint32_t* census;             // optional outputs (see ctaclust.h)
    int32_t* exec_sm;
    int32_t* map;
};

__device__ __forceinline__ int32_t* ws_agent_ctr(const Sched& s) { return s.ws; }
__device__ __forceinline__ int32_t* ws_head(const Sched& s) { return s.ws + s.g.M + 1; }
__device__ __forceinline__ int32_t* ws_gq(const Sched& s) { return s.ws + 2 * s.g.M + 1; }
__device__ __forceinline__ int32_t* ws_done(const Sched& s) { return s.ws + 2 * s.g.M + 2; }
inline size_t ws_ints(int32_t M) { return (size_t)(2 * M + 3); }

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
// relaxed gpu-scope load (no fence, no L1 invalidation)
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

// Queue cursor of one agent (thread 0 only).
struct Cursor {
    int32_t q;        // cluster queue being drained, -1 = finished
    int32_t home;     // first queue scanned
    int32_t scanned;  // queues visited so far
};

// Next order position for this agent or -1.  Own cluster first, then (steal)
// the other clusters round-robin from home.
__device__ __forceinline__ int32_t next_position(const Sched& s, Cursor& c) {
    if (s.mode == MODE_IDENTITY) {
        if (c.q < 0) return -1;
        int32_t v = atom_add_relaxed(ws_gq(s), 1);
        if (v < s.g.V) return v;
        c.q = -1;
        return -1;
    }
    int32_t* head = ws_head(s);
    while (c.q >= 0) {
        int32_t size = cluster_size(s.g, c.q);
        if (ld_relaxed(head + c.q) < size) {
            int32_t w = atom_add_relaxed(head + c.q, 1);
            if (w < size) return cluster_start(s.g, c.q) + w;
        }
        if (!s.steal || ++c.scanned >= s.g.M) { c.q = -1; break; }
        c.q = c.home + c.scanned;
        if (c.q >= s.g.M) c.q -= s.g.M;
    }
    return -1;
}

__device__ __forceinline__ void record(const Sched& s, int32_t v, int32_t lin) {
    if (s.census) atomicAdd(s.census + lin, 1u);
    if (s.exec_sm) s.exec_sm[lin] = (int32_t)smid();
    if (s.map) s.map[v] = lin;
}

// Body concept (all methods called by every thread, with CTA-uniform args):
//   run(bx, by)            one logical CTA of the original kernel
//   prefetch_l2(bx, by)    thread 0 only: warm L2 with the next task's tile
//   finish()               agent is retiring: flush carried state
template <class Body>
__device__ __forceinline__ void agent_loop(const Sched& s, Body& body) {
    __shared__ int32_t s_agent;
    __shared__ int32_t s_next[2];
    Cursor cur_c;
    if (threadIdx.x == 0) {
        // binding: dense SM rank from %smid, agent id by arrival
        uint32_t sm = smid();
        int32_t rank = (int32_t)sm < s.smid_span ? s.rank_of_smid[sm] : -1;
        int32_t arank = rank;                             // rank used for the agent id
        if (rank >= s.g.M) rank = -1;                     // fewer clusters than SMs
        int32_t a = atom_add_relaxed(ws_agent_ctr(s) + (arank < 0 || arank >= s.g.M ? s.g.M : arank), 1);
        // agents with no cluster of their own only steal, from a spread-out start
        cur_c.home = rank >= 0 ? rank : (int32_t)(blockIdx.x % (uint32_t)(s.g.M > 0 ? s.g.M : 1));
        cur_c.scanned = 0;
        cur_c.q = (s.g.V > 0 && s.g.M > 0) ? cur_c.home : -1;
        // throttling (Listing 5 l.20): agents past active_agents retire at once
        const bool active = (a < s.active_agents) && (rank >= 0 || s.steal || s.mode == MODE_IDENTITY);
        if (!active) cur_c.q = -1;
        s_agent = active ? 1 : 0;
        s_next[0] = active ? next_position(s, cur_c) : -1;
    }
    __syncthreads();
    int32_t v = s_next[0];
    int32_t t = 0;
    while (v >= 0) {
        int32_t lin, bx, by;
        lin_to_bxby(s, v, &lin, &bx, &by);
        int32_t nxt = -1;
        int32_t spec_q = -1, spec_w = 0;
        if (threadIdx.x == 0) {
            if (s.prefetch) {
                nxt = next_position(s, cur_c);
                if (nxt >= 0) {
                    int32_t nl, nbx, nby;
                    lin_to_bxby(s, nxt, &nl, &nbx, &nby);
                    body.prefetch_l2(nbx, nby);
                }
            } else if (s.mode == MODE_AGENT && cur_c.q >= 0) {
                // speculative pop: issue the atomic now, look at it after the body
                spec_q = cur_c.q;
                spec_w = atom_add_relaxed(ws_head(s) + spec_q, 1);
            }
        }
        body.run(bx, by);
        if (threadIdx.x == 0) {
            record(s, v, lin);
            if (!s.prefetch) {
                if (spec_q >= 0 && spec_w < cluster_size(s.g, spec_q)) nxt = cluster_start(s.g, spec_q) + spec_w;
                else {
                    if (spec_q >= 0 && cur_c.q == spec_q) {   // own queue ran dry: move on
                        if (!s.steal || ++cur_c.scanned >= s.g.M) cur_c.q = -1;
                        else { cur_c.q = cur_c.home + cur_c.scanned; if (cur_c.q >= s.g.M) cur_c.q -= s.g.M; }
                    }
                    nxt = next_position(s, cur_c);
                }
            }
            s_next[(t + 1) & 1] = nxt;
        }
        __syncthreads();
        v = s_next[(t + 1) & 1];
        ++t;
    }
    if (s_agent) body.finish();
    // the last agent out resets the workspace for the next launch.  Every other
    // agent has consumed the results of all its atomics before arriving here,
    // so no counter can still be in use.
    if (threadIdx.x == 0) {
        int32_t total = (int32_t)(gridDim.x * gridDim.y * gridDim.z);
        if (atom_add_relaxed(ws_done(s), 1) == total - 1) {
            int32_t n = 2 * s.g.M + 2;
            for (int32_t k = 0; k < n; ++k) s.ws[k] = 0;
            *ws_done(s) = 0;
        }
    }
}

// ---- kernels: one per (body, backend) ------------------------------------
template <class Body>
__global__ void __launch_bounds__(Body::kThreads) k_agent(Sched s, typename Body::Params p) {
    Body body(p);
    agent_loop(s, body);
}

template <class Body>
__global__ void __launch_bounds__(Body::kThreads) k_default(Sched s, typename Body::Params p) {
    Body body(p);
    int32_t bx = blockIdx.x, by = blockIdx.y;
    body.run(bx, by);
    if (threadIdx.x == 0) {
        int32_t lin = by * s.g.gx + bx;
        if (s.census) atomicAdd(s.census + lin, 1u);
        if (s.exec_sm) s.exec_sm[lin] = (int32_t)smid();
    }
    body.finish();
}

// Redirection-based clustering (Listing 4, Fig. 9): same number of CTAs as O;
// CTA u runs v = rd_redirect(u).
template <class Body>
__global__ void __launch_bounds__(Body::kThreads) k_redirect(Sched s, typename Body::Params p) {
    Body body(p);
    int32_t u = blockIdx.x;
    int32_t v = rd_redirect(s.g, u);
    int32_t lin, bx, by;
    lin_to_bxby(s, v, &lin, &bx, &by);
    body.run(bx, by);
    if (threadIdx.x == 0) record(s, v, lin);
    body.finish();
}

}  // namespace cc
