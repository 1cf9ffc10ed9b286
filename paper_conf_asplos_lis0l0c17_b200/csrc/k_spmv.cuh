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
// slot per hub column (degree > t, or == t while slots remain), -1 otherwise;
// deg[] is overwritten with the slot id.  ctr[0]: hubs above t, ctr[1]: ties.
__global__ void k_spmv_hot_assign(int32_t* deg, int32_t cols, int32_t t, int32_t n_gt, int32_t max_hot,
                                  int32_t* ctr, int32_t* hot) {
    for (int32_t c = blockIdx.x * blockDim.x + threadIdx.x; c < cols; c += gridDim.x * blockDim.x) {
        const int32_t d = deg[c] < 65535 ? deg[c] : 65535;
        int32_t slot = -1;
        if (d > t && d > 0) slot = atomicAdd(ctr, 1);
        else if (d == t && d > 0) {
            const int32_t e = atomicAdd(ctr + 1, 1);
            if (n_gt + e < max_hot) slot = n_gt + e;
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
        stage_commit(full, lane, 0);
    }

    __device__ __forceinline__ void consume(const Sched& s, int32_t bx, int32_t /*by*/, const uint8_t*, int ctid) {
        __shared__ int32_t s_rowend[SPMV_ROWCAP];
        // products of the CTA's nonzeros, index j stored at j + j/32: the
        // coalesced writes (a warp's 32 consecutive j) are conflict-free, and
        // the merge walk's reads (lane t at ~15 t: its run starts after the
        // rows ended before it) spread over the banks (round 2: j + j/16 put
        // them ~16 words apart -- 41 % excess shared wavefronts, ncu r10l)
        __shared__ float s_prod[SPMV_IPC + SPMV_IPC / 32];
        __shared__ float s_wv[SPMV_THREADS / 32];
        __shared__ int32_t s_wf[SPMV_THREADS / 32];
        const int t = ctid, lane = t & 31, warp = t >> 5;
        const int64_t total = (int64_t)p.rows + p.nnz;
        const int64_t d0 = (int64_t)bx * SPMV_IPC;
        const int64_t d1 = d0 + SPMV_IPC < total ? d0 + SPMV_IPC : total;
        const int32_t x0 = p.part[bx], x1 = p.part[bx + 1];
        const int64_t y0 = d0 - x0, y1 = d1 - x1;
        const int32_t xl = x1 < p.rows ? x1 : p.rows - 1;      // last row to stage
        const bool staged = xl - x0 < SPMV_ROWCAP;
        if (staged)
            for (int32_t i = t; i <= xl - x0; i += kConsumers) s_rowend[i] = p.row_ptr[x0 + i + 1];
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
                    const int32_t j = t + (k0 + k) * kConsumers;
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
                    else xv[k] = ld_hot_issue(p.xh_end + c[k]);
                }
#pragma unroll
                for (int k = 0; k < SPMV_GB; ++k) {
                    const int32_t j = t + (k0 + k) * kConsumers;
                    if (j < nz) s_prod[j + j / 32] = v[k] * xv[k];
                }
            }
        } else if (l2h != 0) {
            // L2 hints (S§8(f)2): col/val streamed (evict_first), x reused (evict_last)
            const bool hf = l2h & L2H_STREAM_FIRST, hl = l2h & L2H_REUSE_LAST;
            const uint64_t pf = l2_evict_first(), pl = l2_evict_last();
#pragma unroll
            for (int k = 0; k < SPMV_IPT; ++k) {
                const int32_t j = t + k * kConsumers;
                if (j < nz) {
                    const int32_t c = hf ? ld_stream_i32_h(p.col + y0 + j, pf) : ld_stream_i32(p.col + y0 + j);
                    const float v = hf ? ld_stream_f32_h(p.val + y0 + j, pf) : ld_stream_f32(p.val + y0 + j);
                    const float* xp = c >= 0 ? p.x + c : p.xh_end + c;
                    s_prod[j + j / 32] = v * (hl ? ld_cached_h(xp, pl) : ld_cached(xp));
                }
            }
        }
        consumer_sync<kConsumers>();
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
                        sum += s_prod[cj + cj / 32];
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
        if (staged) walk(s_rowend);
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
        if (lane == 31) { s_wv[warp] = v; s_wf[warp] = f; }
        consumer_sync<kConsumers>();
        float pv = 0.f;                      // prefix of earlier warps
        for (int w = 0; w < warp; ++w) pv = s_wf[w] ? s_wv[w] : pv + s_wv[w];
        const float T = f ? v : pv + v;      // outgoing carry of this thread
        float incoming = __shfl_up_sync(0xffffffffu, T, 1);
        if (lane == 0) incoming = pv;
        if (t == 0) incoming = 0.f;
        if (has_end) {
            float val = incoming + first_val;
            const bool started_before = (first_row == x0) && (y0 > row_start(x0));
            if (started_before) atomicAdd(p.y + first_row, val);
            else p.y[first_row] = val;
        }
        if (t == kConsumers - 1 && x1 < p.rows && T != 0.f) atomicAdd(p.y + x1, T);
        consumer_sync<kConsumers>();                     // s_wv / s_rowend reuse by the next task
    }
    __device__ __forceinline__ int64_t row_start(int32_t r) const {
        return r == 0 ? 0 : (int64_t)p.row_ptr[r];
    }
    __device__ __forceinline__ void finish(int) {}
};

}  // namespace cc
