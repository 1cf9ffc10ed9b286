// k_spmv.cuh -- CSR SpMV tile body (data-related locality class).
//
// y[i] = sum_{k in [rp[i], rp[i+1])} val[k] * x[col[k]]
//
// Logical CTA b owns the merge-path diagonal range [b*IPC, (b+1)*IPC) of the
// (row ends) x (nonzeros) merge grid, so every logical CTA gets the same number
// of rows + nonzeros however skewed the power-law degree distribution is.  Its
// start coordinate comes from a precomputed table (cc_spmv_partition).  Inside
// the CTA each thread merges IPT items; partial rows are stitched with a
// CTA-wide segmented scan, so at most two atomics per logical CTA touch y
// (the rows it shares with its neighbours); every other row is a plain store.
// The x gathers go through L1 (the data-dependent inter-CTA reuse the paper
// calls hard to exploit); val/col stream past it.
//
// Shared memory is kept small on purpose: on sm_100a L1 and shared memory are
// one 256 KB array per SM, and every KB of smem a resident CTA holds is a KB
// of L1 the R-MAT hub columns of x cannot use.  Row ends are staged only when
// the CTA's row range fits SPMV_ROWCAP (the common case: ~IPC/17 rows at 16
// nnz/row); a CTA over a run of (near-)empty rows reads them from global.
#pragma once
#include "cc_mem.cuh"
#include "cc_runtime.cuh"

namespace cc {

struct SpmvParams {
    int32_t rows; int64_t nnz;
    const int32_t* row_ptr; const int32_t* col; const float* val; const float* x; float* y;
    const int32_t* part;   // part[b] = row coordinate of diagonal b*IPC
    const float* xh_end;   // hub-column form: one past the gathered hub values (col -(k+1) -> xh_end[-(k+1)])
    int32_t n_hot;         // hub slots (0: plain CSR)
};

// Hub gather of the hub-column form (cc_spmv_inspect): xh[n_hot-1-k] = x[hot[k]].
__global__ void k_spmv_hot_gather(const float* __restrict__ x, const int32_t* __restrict__ hot, float* xh,
                                  int32_t n_hot) {
    for (int32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < n_hot; k += gridDim.x * blockDim.x)
        xh[n_hot - 1 - k] = x[hot[k]];
}

// ---- inspector (cc_spmv_inspect) ---------------------------------------------
// references per column
__global__ void k_spmv_col_degree(const int32_t* __restrict__ col, int64_t nnz, int32_t* deg) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nnz; k += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(deg + col[k], 1);
}
// histogram of min(degree, 65535)
__global__ void k_spmv_deg_hist(const int32_t* __restrict__ deg, int32_t cols, int32_t* hist) {
    for (int32_t c = blockIdx.x * blockDim.x + threadIdx.x; c < cols; c += gridDim.x * blockDim.x) {
        const int32_t d = deg[c];
        atomicAdd(hist + (d < 65535 ? d : 65535), 1);
    }
}
// slot per hub column, -1 otherwise; deg[] is overwritten with the slot id.
// Two tiers, each a contiguous slot range: A = [0, T), the T most referenced
// columns (the shared-memory tier of CC_K_SPMV_SHUB), and B = [T, used).  The
// host derives from the degree histogram dA / dB, the degrees of the T-th and
// the used-th most referenced column, n_a = #(degree > dA) and n_b = the
// B columns referenced more than dB times.  Inside a group slots are handed
// out by one atomic counter in the grid-stride column order (warp-aggregated),
// so neighbouring slots hold nearby columns: a row's sorted column run then
// gathers from few lines of the hub array (round 2: degree-ordered or
// scattered slots made the L1 hub form 2-4 % slower).  Degrees clamped at
// 65535; ctr[0..3] zeroed by the host.
__global__ void k_spmv_hot_assign(int32_t* deg, int32_t cols, int32_t dA, int32_t n_a, int32_t T, int32_t dB,
                                  int32_t n_b, int32_t used, int32_t* ctr, int32_t* hot) {
    for (int32_t c = blockIdx.x * blockDim.x + threadIdx.x; c < cols; c += gridDim.x * blockDim.x) {
        const int32_t d = deg[c] < 65535 ? deg[c] : 65535;
        int32_t slot = -1;
        if (used > 0 && d > 0 && d >= dB) {
            if (T > 0 && d > dA) slot = atomicAdd(ctr + 0, 1);                 // tier A, above its threshold
            else {
                int32_t r = -1;                                                // rank among the ties at dA
                if (T > 0 && d == dA) {
                    r = atomicAdd(ctr + 1, 1);
                    if (r < T - n_a) slot = n_a + r;                           // tier A, ties
                }
                if (slot < 0) {
                    if (d > dB) slot = T + atomicAdd(ctr + 2, 1);              // tier B, above its threshold
                    else {                                                     // ties at dB
                        const int32_t q = dA == dB && r >= 0 ? r - (T - n_a) : atomicAdd(ctr + 3, 1);
                        if (T + n_b + q < used) slot = T + n_b + q;
                    }
                }
            }
        }
        deg[c] = slot;
        if (slot >= 0) hot[slot] = c;
    }
}
__global__ void k_spmv_col_encode(const int32_t* __restrict__ col, int64_t nnz, const int32_t* __restrict__ slot,
                                  int32_t* col_hot) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nnz; k += (int64_t)gridDim.x * blockDim.x) {
        const int32_t c = col[k], sl = slot[c];
        col_hot[k] = sl >= 0 ? -(sl + 1) : c;
    }
}

#ifndef CC_SPMV_IPT
#define CC_SPMV_IPT 16
#endif
constexpr int SPMV_IPT = CC_SPMV_IPT;
constexpr int SPMV_THREADS = 256;
constexpr int SPMV_IPC = SPMV_IPT * SPMV_THREADS;   // merge items per logical CTA
constexpr int SPMV_ROWCAP = 512;                    // staged row ends per CTA
#ifndef CC_SPMV_GB
#define CC_SPMV_GB 4
#endif
constexpr int SPMV_GB = CC_SPMV_GB;                 // gathers in flight per thread (batch)
#ifndef CC_SPMV_PREFETCH
#define CC_SPMV_PREFETCH 1
#endif
#ifndef CC_SPMV_MIN_AGENTS
#define CC_SPMV_MIN_AGENTS 5
#endif

// Merge-path search (row ends a[0..a_len) vs natural numbers b[k] = k):
// number of row ends consumed at diagonal d.
__device__ __forceinline__ int64_t merge_search_global(const int32_t* row_end, int64_t a_len,
                                                       int64_t b_len, int64_t d) {
    int64_t lo = d - b_len > 0 ? d - b_len : 0;
    int64_t hi = d < a_len ? d : a_len;
    while (lo < hi) {
        int64_t pv = (lo + hi) >> 1;
        if ((int64_t)row_end[pv] <= d - pv - 1) lo = pv + 1;
        else hi = pv;
    }
    return lo;
}

__global__ void k_spmv_partition(const int32_t* row_ptr, int32_t rows, int64_t nnz,
                                 int32_t nblocks, int32_t* part) {
    int32_t b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b > nblocks) return;
    int64_t total = (int64_t)rows + nnz;
    int64_t d = (int64_t)b * SPMV_IPC;
    if (d > total) d = total;
    part[b] = (int32_t)merge_search_global(row_ptr + 1, rows, nnz, d);
}

// One logical CTA (merge-path block bx) run by one consumer group of
// SPMV_THREADS threads (t = ctid) with its scratch `sc`; hub(c) returns the
// value of hub slot -(c+1) (c < 0, hub-column form).
struct SpmvScratch {
    int32_t* rowend;   // [SPMV_ROWCAP]
    float* prod;       // [SPMV_IPC + SPMV_IPC / 32]
    float* wv;         // [SPMV_THREADS / 32]
    int32_t* wf;       // [SPMV_THREADS / 32]
};
constexpr int SPMV_SCRATCH_BYTES = 4 * (SPMV_ROWCAP + SPMV_IPC + SPMV_IPC / 32 + 2 * (SPMV_THREADS / 32));

template <class HubLd>
__device__ __forceinline__ void spmv_task(const SpmvParams& p, int32_t l2h, int32_t bx, int ctid,
                                          const SpmvScratch& sc, const HubLd& hub) {
    const int t = ctid, lane = t & 31, warp = t >> 5;
    const int64_t total = (int64_t)p.rows + p.nnz;
    const int64_t d0 = (int64_t)bx * SPMV_IPC;
    const int64_t d1 = d0 + SPMV_IPC < total ? d0 + SPMV_IPC : total;
    const int32_t x0 = p.part[bx], x1 = p.part[bx + 1];
    const int64_t y0 = d0 - x0, y1 = d1 - x1;
    const int32_t xl = x1 < p.rows ? x1 : p.rows - 1;      // last row to stage
    const bool staged = xl - x0 < SPMV_ROWCAP;
    if (staged)
        for (int32_t i = t; i <= xl - x0; i += SPMV_THREADS) sc.rowend[i] = p.row_ptr[x0 + i + 1];
    // all products of the CTA, coalesced: val/col stream past L1, the x
    // gathers go through it (16 independent loads per thread in flight)
    const int32_t nz = (int32_t)(y1 - y0);
    if (l2h == 0 && nz > 0) {
        // two phases per batch of SPMV_GB items: all col/val loads in flight,
        // then all x gathers in flight, then the products -- the gathers'
        // latency is paid once per batch, not once per item
#pragma unroll
        for (int k0 = 0; k0 < SPMV_IPT; k0 += SPMV_GB) {
            int32_t c[SPMV_GB];
            float v[SPMV_GB], xv[SPMV_GB];
#pragma unroll
            for (int k = 0; k < SPMV_GB; ++k) {
                const int32_t j = t + (k0 + k) * SPMV_THREADS;
                const bool ok = j < nz;           // past the end: re-read item 0 (nz > 0)
                c[k] = ld_stream_i32_issue(p.col + y0 + (ok ? j : 0));
                v[k] = ld_stream_f32_issue(p.val + y0 + (ok ? j : 0));
            }
#pragma unroll
            for (int k = 0; k < SPMV_GB; ++k) {
                // hub references (negative, hub-column form) read the dense
                // hub array, which stays in L1 (evict_last); every other
                // gather skips L1 (.cg): x has almost no reuse outside the
                // hubs, and L1 then keeps only the hub array (round 2:
                // 1.7 % faster on plain CSR, 4.6 % with 16 K hub slots;
                // profiles/r10/exp/spmv_xcg.json)
                if (c[k] >= 0) xv[k] = ld_l2only_issue(p.x + c[k]);
                else xv[k] = hub(c[k]);
            }
#pragma unroll
            for (int k = 0; k < SPMV_GB; ++k) {
                const int32_t j = t + (k0 + k) * SPMV_THREADS;
                if (j < nz) sc.prod[j + j / 32] = v[k] * xv[k];
            }
        }
    } else if (l2h != 0) {
        // L2 hints (S§8(f)2): col/val streamed (evict_first), x reused (evict_last)
        const bool hf = l2h & L2H_STREAM_FIRST, hl = l2h & L2H_REUSE_LAST;
        const uint64_t pf = l2_evict_first(), pl = l2_evict_last();
#pragma unroll
        for (int k = 0; k < SPMV_IPT; ++k) {
            const int32_t j = t + k * SPMV_THREADS;
            if (j < nz) {
                const int32_t c = hf ? ld_stream_i32_h(p.col + y0 + j, pf) : ld_stream_i32(p.col + y0 + j);
                const float v = hf ? ld_stream_f32_h(p.val + y0 + j, pf) : ld_stream_f32(p.val + y0 + j);
                const float xv = c < 0 ? hub(c) : hl ? ld_cached_h(p.x + c, pl) : ld_cached(p.x + c);
                sc.prod[j + j / 32] = v * xv;
            }
        }
    }
    consumer_sync<SPMV_THREADS>();
    // this thread's start on the merge path, relative to the CTA rectangle
    const int32_t span = (int32_t)(d1 - d0);
    const int32_t dt = t * SPMV_IPT < span ? t * SPMV_IPT : span;
    const int32_t items = span - dt < SPMV_IPT ? span - dt : SPMV_IPT;
    float sum = 0.f, first_val = 0.f;
    int32_t first_row = -1;
    bool has_end = false;
    // search + merge walk over this thread's IPT items; instantiated once
    // with the smem row ends (LDS) and once with the global ones
    auto walk = [&](const int32_t* rowend) {
        int32_t lo = dt - (int32_t)(y1 - y0); if (lo < 0) lo = 0;
        int32_t hi = dt < (x1 - x0) ? dt : (x1 - x0);
        while (lo < hi) {
            int32_t pv = (lo + hi) >> 1;
            if ((int64_t)rowend[pv] <= y0 + dt - pv - 1) lo = pv + 1;
            else hi = pv;
        }
        int32_t cx = x0 + lo;
        int32_t cj = (int32_t)(dt - lo);                 // nonzero index relative to y0
        int32_t re = cx < p.rows ? (int32_t)(rowend[cx - x0] - y0) : INT32_MIN;
#pragma unroll
        for (int it = 0; it < SPMV_IPT; ++it) {
            if (it < items) {
                if (cj < re) {
                    sum += sc.prod[cj + cj / 32];
                    ++cj;
                } else {
                    if (!has_end) { first_row = cx; first_val = sum; has_end = true; }
                    else p.y[cx] = sum;                 // row began and ended in this thread
                    sum = 0.f;
                    ++cx;
                    re = cx < p.rows ? (int32_t)(rowend[cx - x0] - y0) : INT32_MIN;
                }
            }
        }
    };
    if (staged) walk(sc.rowend);
    else walk(p.row_ptr + x0 + 1);
    // segmented inclusive scan of (has_end, carry): T[t] = carry + (has_end ? 0 : T[t-1])
    bool f = has_end;
    float v = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        float vu = __shfl_up_sync(0xffffffffu, v, o);
        int fu = __shfl_up_sync(0xffffffffu, (int)f, o);
        if (lane >= o) { if (!f) v += vu; f = f || fu; }
    }
    if (lane == 31) { sc.wv[warp] = v; sc.wf[warp] = f; }
    consumer_sync<SPMV_THREADS>();
    float pv = 0.f;                      // prefix of earlier warps
    for (int w = 0; w < warp; ++w) pv = sc.wf[w] ? sc.wv[w] : pv + sc.wv[w];
    const float T = f ? v : pv + v;      // outgoing carry of this thread
    float incoming = __shfl_up_sync(0xffffffffu, T, 1);
    if (lane == 0) incoming = pv;
    if (t == 0) incoming = 0.f;
    if (has_end) {
        float val = incoming + first_val;
        const bool started_before = (first_row == x0) && (y0 > (x0 == 0 ? 0 : (int64_t)p.row_ptr[x0]));
        if (started_before) atomicAdd(p.y + first_row, val);
        else p.y[first_row] = val;
    }
    if (t == SPMV_THREADS - 1 && x1 < p.rows && T != 0.f) atomicAdd(p.y + x1, T);
    consumer_sync<SPMV_THREADS>();                     // sc.wv / sc.rowend reuse by the next task
}

// producer side of a task (warp 0): col / val / row_ptr runs of block bx
// from DRAM into L2, one bulk prefetch per lane 0-2
__device__ __forceinline__ void spmv_prefetch(const SpmvParams& p, int32_t bx, int lane) {
    if (CC_SPMV_PREFETCH && lane < 3) {
        const int64_t total = (int64_t)p.rows + p.nnz;
        const int64_t d0 = (int64_t)bx * SPMV_IPC;
        const int64_t d1 = d0 + SPMV_IPC < total ? d0 + SPMV_IPC : total;
        const int32_t x0 = p.part[bx], x1 = p.part[bx + 1];
        const int64_t lo = lane == 2 ? x0 : d0 - x0, hi = lane == 2 ? (int64_t)x1 + 2 : d1 - x1;
        const char* base = lane == 0 ? (const char*)p.col : lane == 1 ? (const char*)p.val
                                                                      : (const char*)p.row_ptr;
        const uintptr_t a0 = ((uintptr_t)(base + 4 * lo)) & ~(uintptr_t)15;
        const uintptr_t a1 = ((uintptr_t)(base + 4 * hi) + 15) & ~(uintptr_t)15;
        if (hi > lo) prefetch_l2_bulk((const void*)a0, (uint32_t)(a1 - a0));
    }
}

struct SpmvBody {
    static constexpr int kConsumers = SPMV_THREADS;
    static constexpr int kStageBytes = 128;       // nothing staged: reads go straight to L1/L2
    static constexpr int kDefaultStages = 2;
    static constexpr int kDefaultBatch = 2;
    static constexpr int kMinAgents = CC_SPMV_MIN_AGENTS;
    static constexpr int kGroups = 1;
    using Params = SpmvParams;
    const SpmvParams& p;
    int32_t l2h = 0;         // cc_l2_hint bits; set by k_agent only (one-shot kernels keep the literal 0)
    __device__ __forceinline__ explicit SpmvBody(const SpmvParams& prm) : p(prm) {}

    // Nothing is staged in smem (it would cost L1, see above).  Instead the
    // producer warp -- in an agent, one or more tasks ahead of the consumers --
    // prefetches the task's col / val runs (and its row_ptr range) from DRAM
    // into L2, so the consumers' streaming loads and the x gathers that depend
    // on them pay one L2 round trip rather than DRAM + L2: the paper's CTA
    // prefetching (section 4.3(III), Listing 5 l.34-37), which the persistent
    // agent's ordered task stream makes possible.
    __device__ __forceinline__ void produce(const Sched&, int32_t bx, int32_t, uint8_t*, uint64_t* full, int lane) {
        spmv_prefetch(p, bx, lane);
        stage_commit(full, lane, 0);
    }

    __device__ __forceinline__ void consume(const Sched&, int32_t bx, int32_t /*by*/, const uint8_t*, int ctid) {
        __shared__ int32_t s_rowend[SPMV_ROWCAP];
        // products of the CTA's nonzeros, index j stored at j + j/32: the
        // coalesced writes (a warp's 32 consecutive j) are conflict-free, and
        // the merge walk's reads (lane t at ~15 t: its run starts after the
        // rows ended before it) spread over the banks (round 2: j + j/16 put
        // them ~16 words apart -- 41 % excess shared wavefronts, ncu r10l)
        __shared__ float s_prod[SPMV_IPC + SPMV_IPC / 32];
        __shared__ float s_wv[SPMV_THREADS / 32];
        __shared__ int32_t s_wf[SPMV_THREADS / 32];
        // hub values from the dense hub array, kept in L1 (evict_last)
        spmv_task(p, l2h, bx, ctid, SpmvScratch{s_rowend, s_prod, s_wv, s_wf},
                  [&](int32_t c) { return ld_hot_issue(p.xh_end + c); });
    }
    __device__ __forceinline__ void finish(int) {}
};


// ---- shared-memory hub tier (CC_K_SPMV_SHUB) ---------------------------------
// The x gathers of SpMV are bound by request throughput (L1 -> L2 requests and
// L2 tag lookups, hottest slice ~95 %: ncu r12a / spmv_m), not by DRAM: each
// gather is its own 32-byte sector.  The hub columns (the most referenced x
// entries, cc_spmv_inspect; slots in non-increasing degree order) are shared
// by every logical CTA -- inter-CTA reuse that a one-shot CTA cannot amortise
// but a persistent agent can: the agent copies the hottest kHubSlots hub
// values into its shared memory ONCE (one bulk copy when its first task is
// staged) and every task it runs reads them with LDS, which never reach the
// L1 tag stage or L2; the remaining hub slots stay in the L1-resident array
// of the plain hub form.  The tier is kept small on purpose: on sm_100a
// shared memory is carved out of L1, and the L1 capacity left over is what
// holds the gathers in flight (round 2: a 43 K-slot tier that filled the SM
// ran 2x slower; 8 K slots with two agents of two groups per SM measured
// best, profiles/r11/exp/spmv_shub_*.json).
#ifndef CC_SHUB_GROUPS
#define CC_SHUB_GROUPS 2
#endif
#ifndef CC_SHUB_AGENTS
#define CC_SHUB_AGENTS 2
#endif
#ifndef CC_SHUB_SLOTS
#define CC_SHUB_SLOTS 8192
#endif
struct SpmvShubBody {
    static constexpr int kConsumers = SPMV_THREADS;
    static constexpr int kGroups = CC_SHUB_GROUPS;
    static constexpr int kMinAgents = CC_SHUB_AGENTS;
    static constexpr int kStageBytes = 128;
    static constexpr int kDefaultStages = 2 * kGroups;
    static constexpr int kDefaultBatch = 2;
    static constexpr int kHubSlots = CC_SHUB_SLOTS;
    // dynamic shared memory after the ring: [kGroups scratch][hub tier (+3: alignment slack)]
    static constexpr int kExtraSmem = kGroups * SPMV_SCRATCH_BYTES + (kHubSlots + 4) * 4;
    using Params = SpmvParams;
    const SpmvParams& p;
    int32_t l2h = 0;
    bool hub_started = false;     // producer: tier copy issued
    bool hub_ready = false;       // consumers: tier copy landed
    __device__ __forceinline__ explicit SpmvShubBody(const SpmvParams& prm) : p(prm) {}

    __device__ __forceinline__ static uint64_t* hub_bar() {
        __shared__ uint64_t bar;
        return &bar;
    }
    __device__ __forceinline__ static uint8_t* extra(const Sched& s) {
        extern __shared__ uint8_t dyn_smem[];
        return ring_base(dyn_smem) + (size_t)s.stages * s.stage_bytes;
    }
    __device__ __forceinline__ float* tier(const Sched& s) const {
        return reinterpret_cast<float*>(extra(s) + kGroups * SPMV_SCRATCH_BYTES);
    }
    // the tier holds xh[a0 .. n_hot) -- slots 0 .. n_hot-a0-1 (xh[n_hot-1-k] is
    // slot k); a0 is 16-byte aligned so that one bulk copy moves it
    __device__ __forceinline__ int32_t tier_first() const {
        const int32_t a = p.n_hot - kHubSlots;
        return a > 0 ? (a & ~3) : 0;
    }

    __device__ __forceinline__ void produce(const Sched& s, int32_t bx, int32_t, uint8_t*, uint64_t* full, int lane) {
        if (!hub_started) {
            // first task of this agent: the tier into shared memory -- bulk
            // copies of the 16-byte part, the (<= 3-float) tail by lane 0
            // before its arrival; the consumers wait on hub_bar once
            hub_started = true;
            if (lane == 0) {
                uint64_t* bar = hub_bar();
                mbar_init(bar, 1);
                fence_mbar_init();
                float* h = tier(s);
                const int32_t a0 = tier_first(), ns = p.n_hot - a0;
                const float* src = p.xh_end - ns;
                const uint32_t nb = ((uint32_t)ns * 4u) & ~15u;
                for (int32_t k = (int32_t)(nb / 4); k < ns; ++k) h[k] = src[k];
                mbar_arrive_tx(bar, nb);
                for (uint32_t off = 0; off < nb; off += 32768u)
                    bulk_g2s(reinterpret_cast<uint8_t*>(h) + off, reinterpret_cast<const uint8_t*>(src) + off,
                             nb - off < 32768u ? nb - off : 32768u, bar);
            }
            __syncwarp();
        }
        spmv_prefetch(p, bx, lane);
        stage_commit(full, lane, 0);
    }

    __device__ __forceinline__ void consume(const Sched& s, int32_t bx, int32_t, const uint8_t*, int ctid) {
        const int g = (int)(threadIdx.x - PRODUCER_THREADS) / kConsumers;
        uint8_t* sb = extra(s) + g * SPMV_SCRATCH_BYTES;
        const SpmvScratch sc{reinterpret_cast<int32_t*>(sb),
                             reinterpret_cast<float*>(sb + 4 * SPMV_ROWCAP),
                             reinterpret_cast<float*>(sb + 4 * (SPMV_ROWCAP + SPMV_IPC + SPMV_IPC / 32)),
                             reinterpret_cast<int32_t*>(sb + 4 * (SPMV_ROWCAP + SPMV_IPC + SPMV_IPC / 32 +
                                                                  SPMV_THREADS / 32))};
        if (!hub_ready) {
            mbar_wait(hub_bar(), 0);
            hub_ready = true;
        }
        const int32_t ns = p.n_hot - tier_first();
        const float* t_end = tier(s) + ns;
        // slot k = -(c+1) < ns: shared-memory tier; the colder slots: the L1 array
        spmv_task(p, l2h, bx, ctid, sc,
                  [&](int32_t c) { return c >= -ns ? t_end[c] : ld_hot_issue(p.xh_end + c); });
    }
    __device__ __forceinline__ void finish(int) {}
};

}  // namespace cc
