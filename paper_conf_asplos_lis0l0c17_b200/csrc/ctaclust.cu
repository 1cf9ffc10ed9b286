// ctaclust.cu -- the C ABI of libctaclust (include/ctaclust.h): planner,
// device binding facts, and the launch dispatcher over the kernel bodies.
#include "../../include/ctaclust.h"

#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <map>
#include <string>
#include <tuple>
#include <vector>

#include "cc_index.cuh"
#include "cc_runtime.cuh"
#include "k_gemv.cuh"
#include "k_atax1.cuh"
#include "k_spmv.cuh"
#include "k_microbench.cuh"
#include "k_hist.cuh"
#include "k_jwave.cuh"
#include "k_stencil.cuh"
#include "k_tbcluster.cuh"

using namespace cc;

// ---------------------------------------------------------------------------
// error plumbing: nothing crosses the ABI but a status and a thread-local text
// ---------------------------------------------------------------------------
static thread_local std::string g_err;
static thread_local int g_cuda_err = 0;

static cc_status fail(cc_status s, const char* fmt, ...) __attribute__((format(printf, 2, 3)));
static cc_status fail(cc_status s, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return s;
}
extern "C" __attribute__((visibility("hidden"))) cc_status cc_internal_fail(cc_status s, const char* msg) {
    return fail(s, "%s", msg);
}
static cc_status cuda_fail(cudaError_t e, const char* what) {
    g_cuda_err = (int)e;
    cudaGetLastError();   // clear sticky-free errors
    return fail(CC_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
}
#define CC_CUDA(call)                                              \
    do {                                                           \
        cudaError_t e_ = (call);                                   \
        if (e_ != cudaSuccess) return cuda_fail(e_, #call);        \
    } while (0)

// ---------------------------------------------------------------------------
// per-device binding facts: SM count, %nsmid span and the dense rank table
// ---------------------------------------------------------------------------
__global__ void k_smid_probe(int32_t* out, int32_t* span, long long spin) {
    if (threadIdx.x == 0) {
        out[blockIdx.x] = (int32_t)smid();
        if (blockIdx.x == 0) *span = (int32_t)nsmid();
        long long t0 = clock64();
        while (clock64() - t0 < spin) {}
    }
}

struct DevFacts {
    bool ready = false;
    int num_sms = 0, smid_span = 0, l2 = 0;
    std::vector<int32_t> rank_of_smid;   // host copy
    int32_t* d_rank = nullptr;           // device copy (never freed: process lifetime)
};
static std::mutex g_dev_mu;
static DevFacts g_dev[64];

static cc_status dev_facts(int device, DevFacts** out) {
    if (device < 0 || device >= 64) return fail(CC_ERR_INVALID_ARG, "device %d out of range", device);
    std::lock_guard<std::mutex> lk(g_dev_mu);
    DevFacts& f = g_dev[device];
    if (f.ready) { *out = &f; return CC_OK; }
    int prev = 0;
    CC_CUDA(cudaGetDevice(&prev));
    CC_CUDA(cudaSetDevice(device));
    CC_CUDA(cudaDeviceGetAttribute(&f.num_sms, cudaDevAttrMultiProcessorCount, device));
    CC_CUDA(cudaDeviceGetAttribute(&f.l2, cudaDevAttrL2CacheSize, device));
    // probe: resident CTAs spinning on every SM record %smid (Listing 3 l.4)
    std::vector<int32_t> seen;
    int32_t span = 0;
    for (int attempt = 0; attempt < 4; ++attempt) {
        int nblk = f.num_sms * (attempt == 0 ? 8 : 16);
        int32_t *d_out = nullptr, *d_span = nullptr;
        CC_CUDA(cudaMalloc(&d_out, sizeof(int32_t) * nblk));
        CC_CUDA(cudaMalloc(&d_span, sizeof(int32_t)));
        k_smid_probe<<<nblk, 32>>>(d_out, d_span, 200000LL << attempt);
        cudaError_t e = cudaDeviceSynchronize();
        std::vector<int32_t> h(nblk);
        if (e == cudaSuccess) e = cudaMemcpy(h.data(), d_out, sizeof(int32_t) * nblk, cudaMemcpyDeviceToHost);
        if (e == cudaSuccess) e = cudaMemcpy(&span, d_span, sizeof(int32_t), cudaMemcpyDeviceToHost);
        cudaFree(d_out);
        cudaFree(d_span);
        if (e != cudaSuccess) return cuda_fail(e, "smid probe");
        seen.insert(seen.end(), h.begin(), h.end());
        std::sort(seen.begin(), seen.end());
        seen.erase(std::unique(seen.begin(), seen.end()), seen.end());
        if ((int)seen.size() >= f.num_sms) break;
    }
    if (span <= 0) span = seen.empty() ? f.num_sms : seen.back() + 1;
    span = std::max(span, seen.empty() ? 0 : seen.back() + 1);
    f.smid_span = span;
    f.rank_of_smid.assign(span, -1);
    for (size_t k = 0; k < seen.size(); ++k) f.rank_of_smid[seen[k]] = (int32_t)k;
    CC_CUDA(cudaMalloc(&f.d_rank, sizeof(int32_t) * span));
    CC_CUDA(cudaMemcpy(f.d_rank, f.rank_of_smid.data(), sizeof(int32_t) * span, cudaMemcpyHostToDevice));
    CC_CUDA(cudaSetDevice(prev));
    f.ready = true;
    *out = &f;
    return CC_OK;
}

// ---------------------------------------------------------------------------
// planner
// ---------------------------------------------------------------------------
struct cc_plan_s {
    Grid g{};
    int device = -1;
    std::vector<int32_t> perm, offsets, user;
    int32_t* d_user = nullptr;
    int32_t* d_ws = nullptr;
    DevFacts* facts = nullptr;
    // workspace ownership: the stream of the last agent launch that used d_ws
    // and an event recorded after it (outside graph capture)
    std::mutex ws_mu;
    cudaStream_t ws_stream = nullptr;
    cudaEvent_t ws_done = nullptr;
    bool ws_pending = false;
};

// The agent backends share the plan's self-resetting workspace (queue heads,
// agent and claim counters).  Two launches in flight at once would interleave
// their queue atomics and break exactly-once coverage, so launches on one plan
// are serialised: under the plan's mutex (held across the launch and the event
// record, so two host threads cannot both pass), a launch on a stream other
// than the previous one's first makes its stream wait for the previous
// launch's completion event (cudaStreamWaitEvent: ordering, no host block).
// Launches captured into a CUDA graph are the caller's to order (no event of
// another stream may be waited on inside a capture); they record nothing.
struct WsLease {
    cc_plan_s* p;
    cudaStream_t st;
    bool capturing = false;
    std::unique_lock<std::mutex> lk;
    cc_status acquire();
    cc_status release();
};
cc_status WsLease::acquire() {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    CC_CUDA(cudaStreamIsCapturing(st, &cs));
    capturing = cs != cudaStreamCaptureStatusNone;
    if (capturing) return CC_OK;
    lk = std::unique_lock<std::mutex>(p->ws_mu);
    if (p->ws_pending && p->ws_stream != st) CC_CUDA(cudaStreamWaitEvent(st, p->ws_done, 0));
    return CC_OK;
}
cc_status WsLease::release() {
    if (capturing) return CC_OK;
    if (!p->ws_done) CC_CUDA(cudaEventCreateWithFlags(&p->ws_done, cudaEventDisableTiming));
    CC_CUDA(cudaEventRecord(p->ws_done, st));
    p->ws_stream = st;
    p->ws_pending = true;
    return CC_OK;
}

extern "C" cc_status cc_plan_create(const cc_plan_desc* d, cc_plan* out) {
    if (!d || !out) return fail(CC_ERR_INVALID_ARG, "null argument");
    *out = nullptr;
    if (d->gx < 0 || d->gy < 0) return fail(CC_ERR_INVALID_ARG, "negative grid");
    if (d->order < CC_ORDER_ROW || d->order > CC_ORDER_USER) return fail(CC_ERR_INVALID_ARG, "bad order %d", d->order);
    if (d->order == CC_ORDER_TILE && (d->tile_w < 1 || d->tile_h < 1))
        return fail(CC_ERR_INVALID_ARG, "tile dims must be >= 1");
    int64_t V = (int64_t)d->gx * (int64_t)d->gy;
    if (V > INT32_MAX) return fail(CC_ERR_OVERFLOW, "gx*gy = %lld exceeds int32", (long long)V);
    if (d->order == CC_ORDER_USER && V > 0 && !d->user_order) return fail(CC_ERR_INVALID_ARG, "USER order needs user_order");
    int M = d->num_clusters;
    DevFacts* facts = nullptr;
    if (d->device >= 0) {
        cc_status s = dev_facts(d->device, &facts);
        if (s != CC_OK) return s;
        if (M == 0) M = facts->num_sms;
    }
    if (M < 1) return fail(CC_ERR_INVALID_ARG, "num_clusters must be >= 1 (or 0 with a device)");
    cc_plan_s* p = new cc_plan_s();
    p->device = d->device;
    p->facts = facts;
    Grid& g = p->g;
    g.gx = d->gx; g.gy = d->gy; g.order = d->order;
    // a tile wider / taller than the grid is the whole grid in that direction
    // (clamped, so the decode's tile products stay inside int32)
    g.tw = d->order == CC_ORDER_TILE ? std::min(d->tile_w, std::max(d->gx, 1)) : 1;
    g.th = d->order == CC_ORDER_TILE ? std::min(d->tile_h, std::max(d->gy, 1)) : 1;
    g.V = (int32_t)V; g.M = M; g.q = (int32_t)(V / M); g.r = (int32_t)(V % M);
    if (d->order == CC_ORDER_USER) {
        p->user.assign(d->user_order, d->user_order + V);
        std::vector<uint8_t> hit(V, 0);
        for (int64_t k = 0; k < V; ++k) {
            int32_t l = p->user[k];
            if (l < 0 || l >= V || hit[l]) { delete p; return fail(CC_ERR_NOT_PERMUTATION, "user_order[%lld] = %d", (long long)k, l); }
            hit[l] = 1;
        }
    }
    // Step 1 + 2: perm[v] = lin of the CTA at order position v.  Clusters are
    // contiguous chunks of the order, so the cluster-major table is the order.
    p->perm.resize(V);
    for (int32_t v = 0; v < (int32_t)V; ++v) {
        if (d->order == CC_ORDER_USER) { p->perm[v] = p->user[v]; continue; }
        int32_t bx, by;
        decode(g, v, &bx, &by);
        p->perm[v] = by * g.gx + bx;
    }
    p->offsets.resize(M + 1);
    for (int i = 0; i <= M; ++i) p->offsets[i] = i < M ? cluster_start(g, i) : g.V;
    if (d->device >= 0) {
        // the tables are filled on a private non-blocking stream and only that
        // stream is synchronised: creating a plan does not wait for (or stall)
        // work queued on the caller's streams
        int prev = 0;
        cudaStream_t ps = nullptr;
        cudaError_t e = cudaGetDevice(&prev);
        if (e == cudaSuccess) e = cudaSetDevice(d->device);
        if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&ps, cudaStreamNonBlocking);
        if (e == cudaSuccess) e = cudaMalloc(&p->d_ws, sizeof(int32_t) * ws_ints(M));
        if (e == cudaSuccess) e = cudaMemsetAsync(p->d_ws, 0, sizeof(int32_t) * ws_ints(M), ps);
        if (e == cudaSuccess && d->order == CC_ORDER_USER && V > 0) {
            e = cudaMalloc(&p->d_user, sizeof(int32_t) * V);
            if (e == cudaSuccess)
                e = cudaMemcpyAsync(p->d_user, p->user.data(), sizeof(int32_t) * V, cudaMemcpyHostToDevice, ps);
        }
        if (e == cudaSuccess) e = cudaStreamSynchronize(ps);
        if (ps) cudaStreamDestroy(ps);
        cudaSetDevice(prev);
        if (e != cudaSuccess) { cudaFree(p->d_ws); cudaFree(p->d_user); delete p; return cuda_fail(e, "plan device tables"); }
    }
    *out = p;
    return CC_OK;
}

extern "C" cc_status cc_plan_destroy(cc_plan p) {
    if (!p) return CC_OK;
    if (p->d_ws) cudaFree(p->d_ws);
    if (p->d_user) cudaFree(p->d_user);
    if (p->ws_done) cudaEventDestroy(p->ws_done);
    delete p;
    return CC_OK;
}

extern "C" cc_status cc_plan_info(cc_plan p, int64_t* V, int32_t* M, int32_t* q, int32_t* r) {
    if (!p) return fail(CC_ERR_INVALID_ARG, "null plan");
    if (V) *V = p->g.V;
    if (M) *M = p->g.M;
    if (q) *q = p->g.q;
    if (r) *r = p->g.r;
    return CC_OK;
}

extern "C" cc_status cc_plan_table(cc_plan p, int32_t* perm, int32_t* offsets) {
    if (!p) return fail(CC_ERR_INVALID_ARG, "null plan");
    if (perm && !p->perm.empty()) memcpy(perm, p->perm.data(), sizeof(int32_t) * p->perm.size());
    if (offsets) memcpy(offsets, p->offsets.data(), sizeof(int32_t) * p->offsets.size());
    return CC_OK;
}

extern "C" cc_status cc_plan_lookup(cc_plan p, int32_t v, int32_t* w, int32_t* i) {
    if (!p || !w || !i) return fail(CC_ERR_INVALID_ARG, "null argument");
    if (v < 0 || v >= p->g.V) return fail(CC_ERR_INVALID_ARG, "v = %d outside [0, %d)", v, p->g.V);
    f_of(p->g, v, w, i);
    return CC_OK;
}

extern "C" cc_status cc_plan_invert(cc_plan p, int32_t w, int32_t i, int32_t* v) {
    if (!p || !v) return fail(CC_ERR_INVALID_ARG, "null argument");
    if (i < 0 || i >= p->g.M || w < 0 || w >= cluster_size(p->g, i))
        return fail(CC_ERR_INVALID_ARG, "(w, i) = (%d, %d) is not a slot", w, i);
    *v = f_inv(p->g, w, i);
    return CC_OK;
}

extern "C" cc_status cc_device_info(int32_t device, int32_t* num_sms, int32_t* smid_span, int32_t* l2) {
    DevFacts* f = nullptr;
    cc_status s = dev_facts(device, &f);
    if (s != CC_OK) return s;
    if (num_sms) *num_sms = f->num_sms;
    if (smid_span) *smid_span = f->smid_span;
    if (l2) *l2 = f->l2;
    return CC_OK;
}

extern "C" cc_status cc_sm_rank_table(int32_t device, int32_t* rank, int32_t cap, int32_t* span) {
    DevFacts* f = nullptr;
    cc_status s = dev_facts(device, &f);
    if (s != CC_OK) return s;
    if (span) *span = f->smid_span;
    if (rank) {
        if (cap < f->smid_span) return fail(CC_ERR_INVALID_ARG, "capacity %d < smid span %d", cap, f->smid_span);
        memcpy(rank, f->rank_of_smid.data(), sizeof(int32_t) * f->smid_span);
    }
    return CC_OK;
}

// ---------------------------------------------------------------------------
// launch
// ---------------------------------------------------------------------------
extern "C" cc_status cc_launch_opts_default(cc_launch_opts* o) {
    if (!o) return fail(CC_ERR_INVALID_ARG, "null opts");
    memset(o, 0, sizeof *o);
    o->backend = CC_BACKEND_AGENT;
    o->steal = 1;
    o->cluster_size = 2;
    o->stages = 0;
    o->batch = 0;
    o->l2_hint = 0;
    o->carveout = -1;
    return CC_OK;
}

#define CC_TRY(...) do { cc_status s_ = (__VA_ARGS__); if (s_ != CC_OK) return s_; } while (0)

// switches to a device and back on scope exit (every return path of cc_launch)
struct DeviceGuard {
    int prev = -1;
    bool switched = false;
    cc_status set(int dev) {
        CC_CUDA(cudaGetDevice(&prev));
        if (prev != dev) {
            CC_CUDA(cudaSetDevice(dev));
            switched = true;
        }
        return CC_OK;
    }
    ~DeviceGuard() {
        if (switched) cudaSetDevice(prev);
    }
};

static inline int32_t cdiv(int64_t a, int64_t b) { return (int32_t)((a + b - 1) / b); }
static inline bool al16(const void* p) { return ((uintptr_t)p & 15) == 0; }

extern "C" cc_status cc_kernel_grid(int32_t k, const void* a, int32_t* gx, int32_t* gy) {
    if (!a || !gx || !gy) return fail(CC_ERR_INVALID_ARG, "null argument");
    switch (k) {
    case CC_K_CENSUS: { auto* c = (const cc_census_args*)a; *gx = c->gx; *gy = c->gy; return CC_OK; }
    case CC_K_MATVEC: { auto* c = (const cc_matvec_args*)a; *gx = cdiv(c->n, 32); *gy = cdiv(c->m, 32); return CC_OK; }
    case CC_K_ATAX: { auto* c = (const cc_atax_args*)a; *gx = cdiv(c->n, 256); *gy = cdiv(c->m, 32); return CC_OK; }
    case CC_K_ATAX_FUSED: { auto* c = (const cc_atax_args*)a; *gx = c->m > 0 ? 1 : 0; *gy = c->m; return CC_OK; }
    case CC_K_BICG: { auto* c = (const cc_bicg_args*)a; *gx = cdiv(c->n, 256); *gy = cdiv(c->m, 32); return CC_OK; }
    case CC_K_MVT: { auto* c = (const cc_mvt_args*)a; *gx = cdiv(c->n, 256); *gy = cdiv(c->m, 32); return CC_OK; }
    case CC_K_JACOBI5: {
        auto* c = (const cc_jacobi5_args*)a;
        if (c->row_lo != 0 || c->row_hi != 0) {
            if (c->row_lo < 0 || c->row_hi <= c->row_lo || c->row_hi > c->rows)
                return fail(CC_ERR_INVALID_ARG, "jacobi5 row window [%d, %d) outside [0, %d]", c->row_lo, c->row_hi, c->rows);
            *gx = cdiv(c->cols, 32); *gy = cdiv(c->row_hi - c->row_lo, 32); return CC_OK;
        }
        *gx = cdiv(c->cols, 32); *gy = cdiv(c->rows, 32); return CC_OK;
    }
    case CC_K_JACOBI5_HALO: { auto* c = (const cc_jacobi5_halo_args*)a; *gx = cdiv(c->cols, 32); *gy = cdiv(c->rows, 32); return CC_OK; }
    case CC_K_JACOBI5_WAVE: {
        auto* c = (const cc_jacobi5_args*)a;
        if (c->fuse < 0 || c->fuse > 8) return fail(CC_ERR_INVALID_ARG, "jacobi5_wave: fuse %d outside [0, 8]", c->fuse);
        const int K = c->fuse < 1 ? 1 : c->fuse;
        const int T = c->tile_rows == 0 ? JW_ROWS : c->tile_rows;
        if (T < 8 || T > 1024) return fail(CC_ERR_INVALID_ARG, "jacobi5_wave: tile_rows %d outside [8, 1024]", c->tile_rows);
        *gx = cdiv(c->cols, jw_strip_cols(jw_halo_chunks(K))); *gy = cdiv(c->rows, T); return CC_OK;
    }
    case CC_K_CONV2D: { auto* c = (const cc_conv2d_args*)a; *gx = cdiv(c->cols, 32); *gy = cdiv(c->rows, 32); return CC_OK; }
    case CC_K_SPMV: case CC_K_SPMV_SHUB: {
        auto* c = (const cc_spmv_args*)a;
        int64_t b = ((int64_t)c->rows + c->nnz + SPMV_IPC - 1) / SPMV_IPC;
        if (b > INT32_MAX - 1) return fail(CC_ERR_OVERFLOW, "spmv grid");
        *gx = (int32_t)b; *gy = 1; return CC_OK;
    }
    case CC_K_HIST64: {
        auto* c = (const cc_hist64_args*)a;
        if (c->n < 0 || c->n > (int64_t)UINT32_MAX) return fail(CC_ERR_INVALID_ARG, "hist64: n %lld outside [0, 2^32)", (long long)c->n);
        *gx = cdiv(c->n, HIST_CHUNK); *gy = 1; return CC_OK;
    }
    default: return fail(CC_ERR_INVALID_ARG, "unknown kernel %d", k);
    }
}

struct CensusParams { int32_t dummy; };
struct CensusBody {   // empty body: binding, queues and census only
    static constexpr int kConsumers = 32;
    static constexpr int kStageBytes = 128;
    static constexpr int kDefaultStages = 2;
    static constexpr int kDefaultBatch = 1;
    static constexpr int kMinAgents = 8;
    static constexpr int kGroups = 1;
    using Params = CensusParams;
    int32_t l2h = 0;
    __device__ __forceinline__ explicit CensusBody(const CensusParams&) {}
    __device__ __forceinline__ void produce(const Sched&, int32_t, int32_t, uint8_t*, uint64_t* full, int lane) { stage_commit(full, lane, 0); }
    __device__ __forceinline__ void consume(const Sched&, int32_t, int32_t, const uint8_t*, int) {}
    __device__ __forceinline__ void finish(int) {}
};

using MatvecB = GemvBody<32, 32, true, false>;
using RowB = GemvBody<32, 256, true, false>;
using ColB = GemvBody<32, 256, false, true>;
using BothB = GemvBody<32, 256, true, true>;

// the header's tier size is the shipped build's
static_assert(SpmvShubBody::kHubSlots == CC_SPMV_SHUB_SLOTS || CC_SHUB_SLOTS != 8192,
              "include/ctaclust.h CC_SPMV_SHUB_SLOTS out of date");

// bytes a body keeps in dynamic shared memory after its ring (kExtraSmem)
template <class B, class = void> struct ExtraSmem { static constexpr int value = 0; };
template <class B> struct ExtraSmem<B, decltype((void)B::kExtraSmem)> { static constexpr int value = B::kExtraSmem; };

template <class Body>
static size_t dyn_smem(int stages, bool direct = false) {
    // direct loads stage nothing: keep the ring minimal so L1 keeps the space
    // (bodies whose direct path needs a per-task buffer size it themselves)
    return (size_t)stages * (direct ? direct_stage_bytes<Body>() : Body::kStageBytes) + 128 + ExtraSmem<Body>::value;
}

// Opt every instantiation of a body into large dynamic shared memory once.
template <class Body>
static cc_status prepare_body(int device) {
    static std::mutex mu;
    static bool done[64] = {false};
    std::lock_guard<std::mutex> lk(mu);
    if (device < 0 || device >= 64) return fail(CC_ERR_INVALID_ARG, "device");
    if (!done[device]) {
        int optin = 0;
        CC_CUDA(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, device));
        cudaFuncAttributes fa{};
        CC_CUDA(cudaFuncGetAttributes(&fa, k_agent<Body>));
        const int mx = (int)std::min(dyn_smem<Body>(MAX_STAGES), (size_t)(optin - (int)fa.sharedSizeBytes));
        const int one = (int)dyn_smem<Body>(1);
        CC_CUDA(cudaFuncSetAttribute(k_agent<Body>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx));
        CC_CUDA(cudaFuncSetAttribute(k_static<Body>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx));
        CC_CUDA(cudaFuncSetAttribute(k_default<Body>, cudaFuncAttributeMaxDynamicSharedMemorySize, one));
        CC_CUDA(cudaFuncSetAttribute(k_redirect<Body>, cudaFuncAttributeMaxDynamicSharedMemorySize, one));
        done[device] = true;
    }
    return CC_OK;
}

// agents per SM the hardware can keep resident for `stages` ring buffers
template <class Body>
static cc_status occupancy(int device, int stages, int* occ, bool direct = false) {
    CC_TRY(prepare_body<Body>(device));
    static std::mutex mu;
    static int cache[64][MAX_STAGES + 1][2] = {};
    std::lock_guard<std::mutex> lk(mu);
    if (stages < 1 || stages > MAX_STAGES) return fail(CC_ERR_INVALID_ARG, "stages %d outside [1, %d]", stages, MAX_STAGES);
    if (!cache[device][stages][direct]) {
        int prev = 0, n = 0;
        CC_CUDA(cudaGetDevice(&prev));
        CC_CUDA(cudaSetDevice(device));
        CC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_agent<Body>, Body::kGroups * Body::kConsumers + PRODUCER_THREADS,
                                                              dyn_smem<Body>(stages, direct)));
        CC_CUDA(cudaSetDevice(prev));
        cache[device][stages][direct] = n > 0 ? n : -1;
    }
    *occ = cache[device][stages][direct];
    if (*occ < 0) return fail(CC_ERR_UNSUPPORTED, "%d stages of %d bytes do not fit one SM", stages, Body::kStageBytes);
    return CC_OK;
}

template <class B> static cc_status jw_occupancy(int device, int* warps);

extern "C" cc_status cc_max_agents(int32_t k, int32_t device, int32_t* out) {
    if (!out) return fail(CC_ERR_INVALID_ARG, "null out");
    int occ = 0;
    cc_status s;
    switch (k) {
    case CC_K_CENSUS: s = occupancy<CensusBody>(device, CensusBody::kDefaultStages, &occ); break;
    case CC_K_MATVEC: s = occupancy<MatvecB>(device, MatvecB::kDefaultStages, &occ); break;
    case CC_K_ATAX: s = occupancy<RowB>(device, RowB::kDefaultStages, &occ); break;
    case CC_K_ATAX_FUSED: s = occupancy<AtaxFusedBody>(device, AtaxFusedBody::kDefaultStages, &occ); break;
    case CC_K_BICG: case CC_K_MVT: s = occupancy<BothB>(device, BothB::kDefaultStages, &occ); break;
    case CC_K_JACOBI5: s = occupancy<Jacobi5Body>(device, Jacobi5Body::kDefaultStages, &occ); break;
    case CC_K_JACOBI5_HALO: s = occupancy<Jacobi5HaloBody>(device, Jacobi5HaloBody::kDefaultStages, &occ); break;
    case CC_K_JACOBI5_WAVE: s = jw_occupancy<JwJacobi<4, 1>>(device, &occ); break;
    case CC_K_CONV2D: s = occupancy<Conv2dBody<3>>(device, Conv2dBody<3>::kDefaultStages, &occ); break;
    case CC_K_SPMV: s = occupancy<SpmvBody>(device, SpmvBody::kDefaultStages, &occ); break;
    case CC_K_SPMV_SHUB: s = occupancy<SpmvShubBody>(device, SpmvShubBody::kDefaultStages, &occ); break;
    case CC_K_HIST64: s = occupancy<HistBody>(device, HistBody::kDefaultStages, &occ); break;
    default: return fail(CC_ERR_INVALID_ARG, "unknown kernel %d", k);
    }
    if (s == CC_OK) *out = occ;
    return s;
}

// Preferred L1/shared carveout of one kernel function (cc_launch_opts.carveout);
// the attribute is per function and sticky, so it is set only when it changes.
template <class K>
static cc_status set_carveout(K* fn, int32_t pct) {
    static std::mutex mu;
    static std::map<const void*, int32_t> cur;
    std::lock_guard<std::mutex> lk(mu);
    auto it = cur.find((const void*)fn);
    const int32_t have = it == cur.end() ? -1 : it->second;
    if (have == pct) return CC_OK;
    CC_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, pct));
    cur[(const void*)fn] = pct;
    return CC_OK;
}

struct LaunchCtx {
    cc_plan p;
    const cc_launch_opts* o;
    cudaStream_t st;
    int32_t* nl;
};

// Ring depth of an agent launch: the requested stages rounded UP to a
// multiple of the body's consumer groups.  Group g consumes tasks g, g+G, ...,
// i.e. slots (g + kG) mod S; with S % G == 0 every slot belongs to one group,
// so a group's successive waits on a slot are for consecutive phases.  With
// S % G != 0 two groups share a slot, and a group can reach its wait for a
// slot while the other group's fill of it is still in flight -- the
// one-bit phase parity then reports the phase two back as complete and the
// group consumes the wrong task (round 2: stages = 3 with two groups hung or
// faulted on full-size stencils; scripts/probe_stages.py).
template <class Body>
static int ring_depth(int requested) {
    int S = requested > 0 ? requested : Body::kDefaultStages;
    S = ((S + Body::kGroups - 1) / Body::kGroups) * Body::kGroups;
    return S < MAX_STAGES ? S : MAX_STAGES - MAX_STAGES % Body::kGroups;
}

template <class Body>
static cc_status launch_body(const LaunchCtx& c, const typename Body::Params& prm) {
    const Grid& g = c.p->g;
    if (g.V == 0) return CC_OK;
    const cc_launch_opts& o = *c.o;
    CC_TRY(prepare_body<Body>(c.p->device));
    Sched s{};
    s.g = g;
    s.user = c.p->d_user;
    s.rank_of_smid = c.p->facts->d_rank;
    s.smid_span = c.p->facts->smid_span;
    s.ws = c.p->d_ws;
    s.steal = o.steal;
    s.batch = o.batch > 0 ? o.batch : Body::kDefaultBatch;
    s.staging = o.staging == CC_STAGING_DEFAULT ? CC_STAGING_TMA : o.staging;
    s.l2_hint = o.l2_hint;
    const bool direct = s.staging == CC_STAGING_DIRECT;
    s.stage_bytes = direct ? (uint32_t)direct_stage_bytes<Body>() : (uint32_t)Body::kStageBytes;
    s.census = o.d_census;
    s.exec_sm = o.d_exec_sm;
    s.map = o.d_map;
    const int threads = Body::kConsumers + PRODUCER_THREADS;
    switch (o.backend) {
    case CC_BACKEND_DEFAULT: {
        if (g.gy > 65535) return fail(CC_ERR_UNSUPPORTED, "default backend: gy %d > 65535", g.gy);
        CC_TRY(set_carveout(k_default<Body>, o.carveout));
        s.map = nullptr;
        s.stages = 1;
        k_default<Body><<<dim3(g.gx, g.gy), threads, dyn_smem<Body>(1, direct), c.st>>>(s, prm);
        break;
    }
    case CC_BACKEND_REDIRECT:
        CC_TRY(set_carveout(k_redirect<Body>, o.carveout));
        s.stages = 1;
        k_redirect<Body><<<g.V, threads, dyn_smem<Body>(1, direct), c.st>>>(s, prm);
        break;
    case CC_BACKEND_AGENT:
    case CC_BACKEND_AGENT_IDENTITY: {
        int S = ring_depth<Body>(o.stages);
        int occ = 0;
        CC_TRY(set_carveout(k_agent<Body>, o.carveout));
        if (o.carveout < 0) CC_TRY(occupancy<Body>(c.p->device, S, &occ, direct));
        else {
            CC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_agent<Body>,
                                                                  Body::kGroups * Body::kConsumers + PRODUCER_THREADS,
                                                                  dyn_smem<Body>(S, direct)));
            if (occ < 1) return fail(CC_ERR_UNSUPPORTED, "carveout %d leaves no room for one agent", o.carveout);
        }
        const int maxa = o.max_agents > 0 ? std::min(o.max_agents, occ) : occ;
        s.active_agents = o.active_agents > 0 ? std::min(o.active_agents, maxa) : maxa;
        s.throttle = s.active_agents < maxa;
        s.mode = o.backend == CC_BACKEND_AGENT ? MODE_AGENT : MODE_IDENTITY;
        s.stages = S;
        const int grid = c.p->facts->num_sms * maxa;
        WsLease lease{c.p, c.st};
        CC_TRY(lease.acquire());
        k_agent<Body><<<grid, Body::kGroups * Body::kConsumers + PRODUCER_THREADS, dyn_smem<Body>(S, direct), c.st>>>(s, prm);
        if (cudaPeekAtLastError() == cudaSuccess) CC_TRY(lease.release());
        break;
    }
    case CC_BACKEND_AGENT_STATIC: {
        int S = ring_depth<Body>(o.stages);
        CC_TRY(set_carveout(k_static<Body>, o.carveout));
        s.active_agents = 1;
        s.throttle = 0;
        s.steal = 0;
        s.mode = MODE_STATIC;
        s.stages = S;
        k_static<Body><<<g.M, Body::kGroups * Body::kConsumers + PRODUCER_THREADS, dyn_smem<Body>(S, direct), c.st>>>(s, prm);
        break;
    }
    default:
        return fail(CC_ERR_UNSUPPORTED, "backend %d not available for this kernel", o.backend);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "kernel launch");
    if (c.nl) ++*c.nl;
    return CC_OK;
}

// ---- CC_K_JACOBI5_WAVE: warp agents (k_jwave.cuh) -------------------------
// opt the kernel into its dynamic shared memory (once per device)
template <class B, int KIND>
static cc_status jw_prepare(int device) {
    static std::mutex mu;
    static bool done[64] = {false};
    if (device < 0 || device >= 64) return fail(CC_ERR_INVALID_ARG, "device");
    std::lock_guard<std::mutex> lk(mu);
    if (!done[device]) {
        CC_CUDA(cudaFuncSetAttribute(k_strip<B, KIND>, cudaFuncAttributeMaxDynamicSharedMemorySize, jw_smem<B>(KIND)));
        done[device] = true;
    }
    return CC_OK;
}

// worker warps per SM the hardware keeps resident
template <class B>
static cc_status jw_occupancy(int device, int* warps) {
    static std::mutex mu;
    static int cache[64] = {};
    if (device < 0 || device >= 64) return fail(CC_ERR_INVALID_ARG, "device");
    std::lock_guard<std::mutex> lk(mu);
    if (!cache[device]) {
        int prev = 0, n = 0;
        CC_CUDA(cudaGetDevice(&prev));
        CC_CUDA(cudaSetDevice(device));
        cc_status st = jw_prepare<B, JW_DYNAMIC>(device);
        if (st == CC_OK)
            CC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_strip<B, JW_DYNAMIC>, jw_threads<B>(JW_DYNAMIC),
                                                                  jw_smem<B>(JW_DYNAMIC)));
        CC_CUDA(cudaSetDevice(prev));
        if (st != CC_OK) return st;
        cache[device] = n > 0 ? n * jw_workers<B>(JW_DYNAMIC) : -1;
    }
    *warps = cache[device];
    if (*warps < 0) return fail(CC_ERR_UNSUPPORTED, "strip kernel: no resident CTA");
    return CC_OK;
}

// one launch of a strip kernel (CC_K_JACOBI5_WAVE): warp agents
template <class B>
static cc_status strip_launch(const LaunchCtx& c, const typename B::Params& prm) {
    const Grid& g = c.p->g;
    if (g.V == 0) return CC_OK;
    const cc_launch_opts& o = *c.o;
    Sched s{};
    s.g = g;
    s.user = c.p->d_user;
    s.rank_of_smid = c.p->facts->d_rank;
    s.smid_span = c.p->facts->smid_span;
    s.ws = c.p->d_ws;
    s.steal = o.steal;
    s.batch = o.batch > 0 ? o.batch : JW_BATCH;
    s.stages = 1;
    // (L2 eviction hints on the row loads / stores measured no gain and cost
    // the row loop registers: not supported here, r15)
    s.census = o.d_census;
    s.exec_sm = o.d_exec_sm;
    s.map = o.d_map;
    switch (o.backend) {
    case CC_BACKEND_DEFAULT:                       // hardware order: warp w of the grid = logical CTA w
        CC_TRY(jw_prepare<B, JW_ONESHOT>(c.p->device));
        CC_TRY(set_carveout(k_strip<B, JW_ONESHOT>, o.carveout));
        s.map = nullptr;
        k_strip<B, JW_ONESHOT><<<cdiv(g.V, jw_workers<B>(JW_ONESHOT)), jw_threads<B>(JW_ONESHOT),
                                  jw_smem<B>(JW_ONESHOT), c.st>>>(s, prm);
        break;
    case CC_BACKEND_AGENT:
    case CC_BACKEND_AGENT_IDENTITY: {
        int occ = 0;
        CC_TRY(set_carveout(k_strip<B, JW_DYNAMIC>, o.carveout));
        CC_TRY(jw_occupancy<B>(c.p->device, &occ));
        const int maxa = o.max_agents > 0 ? std::min(o.max_agents, occ) : occ;
        constexpr int nw = jw_workers<B>(JW_DYNAMIC);
        const int ctas = (maxa + nw - 1) / nw;                         // per SM (workers + a scheduler each)
        const int launched = ctas * nw;
        s.active_agents = o.active_agents > 0 ? std::min(o.active_agents, launched) : launched;
        s.throttle = s.active_agents < launched;
        s.mode = o.backend == CC_BACKEND_AGENT ? MODE_AGENT : MODE_IDENTITY;
        WsLease lease{c.p, c.st};
        CC_TRY(lease.acquire());
        k_strip<B, JW_DYNAMIC><<<c.p->facts->num_sms * ctas, jw_threads<B>(JW_DYNAMIC), jw_smem<B>(JW_DYNAMIC),
                                  c.st>>>(s, prm);
        if (cudaPeekAtLastError() == cudaSuccess) CC_TRY(lease.release());
        break;
    }
    case CC_BACKEND_AGENT_STATIC:                  // worker warp i runs cluster i (Eq. 7 order)
        CC_TRY(jw_prepare<B, JW_STATIC>(c.p->device));
        CC_TRY(set_carveout(k_strip<B, JW_STATIC>, o.carveout));
        s.active_agents = 1;
        s.steal = 0;
        s.mode = MODE_STATIC;
        k_strip<B, JW_STATIC><<<cdiv(g.M, jw_workers<B>(JW_STATIC)), jw_threads<B>(JW_STATIC), jw_smem<B>(JW_STATIC),
                                 c.st>>>(s, prm);
        break;
    default:
        return fail(CC_ERR_UNSUPPORTED, "backend %d not available for the strip kernels", o.backend);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "kernel launch");
    if (c.nl) ++*c.nl;
    return CC_OK;
}

template <int HL>
static cc_status jw_launch(const LaunchCtx& c, const JWaveParams& prm, int K) {
    switch (K) {
    case 1: return strip_launch<JwJacobi<1, HL>>(c, prm);
    case 2: return strip_launch<JwJacobi<2, HL>>(c, prm);
    case 3: return strip_launch<JwJacobi<3, HL>>(c, prm);
    case 4: return strip_launch<JwJacobi<4, HL>>(c, prm);
    default: break;
    }
    if constexpr (HL == 2) {
        switch (K) {
        case 5: return strip_launch<JwJacobi<5, 2>>(c, prm);
        case 6: return strip_launch<JwJacobi<6, 2>>(c, prm);
        case 7: return strip_launch<JwJacobi<7, 2>>(c, prm);
        case 8: return strip_launch<JwJacobi<8, 2>>(c, prm);
        default: break;
        }
    }
    return fail(CC_ERR_INVALID_ARG, "jacobi5_wave: %d sweeps per launch with %d halo chunks", K, HL);
}

// ---- thread-block-cluster backend (conv2d) --------------------------------
static PFN_cuTensorMapEncodeTiled_v12000 tmap_encoder() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        cudaDriverEntryPointQueryResult q;
        void* f = nullptr;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (PFN_cuTensorMapEncodeTiled_v12000)f;
    });
    return fn;
}

// Encoded tensor maps are cached per (base, shape, leading dim, box): a
// 100-sweep Jacobi call encodes each of its two ping-pong buffers once, not
// once per sweep (the encode is ~1-2 us of host time per map).
struct TmapKey {
    const void* base; int32_t rows, cols; int64_t ld; int32_t bc, br;
    bool operator<(const TmapKey& o) const {
        return std::tie(base, rows, cols, ld, bc, br) < std::tie(o.base, o.rows, o.cols, o.ld, o.bc, o.br);
    }
};
static cc_status make_tmap_uncached(CUtensorMap* m, const float* base, int32_t rows, int32_t cols, int64_t ld,
                                    int box_cols, int box_rows);
static cc_status make_tmap(CUtensorMap* m, const float* base, int32_t rows, int32_t cols, int64_t ld, int box_cols,
                           int box_rows) {
    static std::mutex mu;
    static std::map<TmapKey, CUtensorMap> cache;
    const TmapKey k{base, rows, cols, ld, box_cols, box_rows};
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = cache.find(k);
        if (it != cache.end()) { *m = it->second; return CC_OK; }
    }
    CC_TRY(make_tmap_uncached(m, base, rows, cols, ld, box_cols, box_rows));
    std::lock_guard<std::mutex> lk(mu);
    if (cache.size() >= 1024) cache.clear();
    cache[k] = *m;
    return CC_OK;
}
static cc_status make_tmap_uncached(CUtensorMap* m, const float* base, int32_t rows, int32_t cols, int64_t ld,
                                    int box_cols, int box_rows) {
    auto enc = tmap_encoder();
    if (!enc) return fail(CC_ERR_UNSUPPORTED, "cuTensorMapEncodeTiled unavailable");
    cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
    cuuint64_t strides[1] = {(cuuint64_t)ld * 4};
    cuuint32_t box[2] = {(cuuint32_t)box_cols, (cuuint32_t)box_rows};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void*)base, dims, strides, box, estr,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return fail(CC_ERR_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
    return CC_OK;
}

// the four boxes of CC_L2_HINT_HALO_LAST split staging (k_stencil.cuh SplitMaps)
static cc_status make_split(SplitMaps* m, const float* base, int32_t rows, int32_t cols, int64_t ld, int H) {
    CC_TRY(make_tmap(&m->t, base, rows, cols, ld, ST_COLS, 32));
    CC_TRY(make_tmap(&m->b, base, rows, cols, ld, ST_COLS, 2 * H));
    CC_TRY(make_tmap(&m->t2, base, rows, cols, ld, ST_COLS2, 32));
    CC_TRY(make_tmap(&m->b2, base, rows, cols, ld, ST_COLS2, 2 * H));
    return CC_OK;
}

template <int R>
static cc_status launch_tbc(const LaunchCtx& c, const ConvParams<R>& prm) {
    const Grid& g = c.p->g;
    if (g.V == 0) return CC_OK;
    const int C = c.o->cluster_size;
    if (C != 1 && C != 2 && C != 4 && C != 8) return fail(CC_ERR_INVALID_ARG, "cluster_size %d (1, 2, 4 or 8)", C);
    using G = TbcGeom<R, tbc_tw<R>()>;
    CUtensorMap m_c, m_b, m_f;
    CC_TRY(make_tmap(&m_c, prm.in, prm.rows, prm.cols, prm.ld, G::kCols, 32));
    CC_TRY(make_tmap(&m_b, prm.in, prm.rows, prm.cols, prm.ld, G::kCols, G::kHb));
    CC_TRY(make_tmap(&m_f, prm.in, prm.rows, prm.cols, prm.ld, G::kCols, 32 + G::kHb));
    Sched s{};
    s.g = g;
    s.census = c.o->d_census;
    s.exec_sm = c.o->d_exec_sm;
    const size_t smem = tbc_smem_bytes<R>();
    CC_CUDA(cudaFuncSetAttribute(k_conv_tbc<R>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    CC_CUDA(cudaFuncSetAttribute(k_conv_tbc<R>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3(tbc_threads<R>());
    cfg.dynamicSmemBytes = smem;
    cfg.stream = c.st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = C;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = C > 1 ? 1 : 0;                // C = 1: a plain launch (implicit 1-CTA clusters)
    // persistent: as many clusters as can be co-resident (not more than units)
    const int TW = tbc_tw<R>();
    const long units = (long)((g.gx + TW - 1) / TW) * ((g.gy + C - 1) / C);
    cfg.gridDim = dim3(C);
    int nc = 0;
    if (C > 1) {
        CC_CUDA(cudaOccupancyMaxActiveClusters(&nc, k_conv_tbc<R>, &cfg));
    } else {
        CC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nc, k_conv_tbc<R>, tbc_threads<R>(), smem));
        nc *= c.p->facts->num_sms;
    }
    if (nc < 1) return fail(CC_ERR_UNSUPPORTED, "tbcluster: no cluster of %d fits", C);
    if (nc > units) nc = (int)units;
    cfg.gridDim = dim3(nc * C);
    CC_CUDA(cudaLaunchKernelEx(&cfg, k_conv_tbc<R>, m_c, m_b, m_f, s, prm, (int32_t)C));
    if (c.nl) ++*c.nl;
    return CC_OK;
}

template <int TR, int TC>
static cc_status gemv_params(GemvParams* P, const float* A, int64_t lda, int32_t m, int32_t n, const float* vc,
                             const float* vr, float* out_r, float* out_c) {
    memset(P, 0, sizeof *P);
    P->A = A; P->lda = lda; P->m = m; P->n = n; P->vc = vc; P->vr = vr; P->out_r = out_r; P->out_c = out_c;
    if (m > 0 && n > 0) CC_TRY(make_tmap(&P->tmap, A, m, n, lda, TC, TR));
    return CC_OK;
}

static cc_status check_mat(const float* A, int64_t lda, int32_t m, int32_t n) {
    if (m < 0 || n < 0) return fail(CC_ERR_INVALID_ARG, "negative size");
    if ((int64_t)m * n > 0 && !A) return fail(CC_ERR_INVALID_ARG, "null matrix");
    if (lda < n || lda % 4) return fail(CC_ERR_INVALID_ARG, "lda %lld must be >= n and a multiple of 4", (long long)lda);
    if (!al16(A)) return fail(CC_ERR_INVALID_ARG, "matrix not 16-byte aligned");
    return CC_OK;
}
static cc_status check_vec(const void* v, int64_t len, const char* name) {
    if (len > 0 && !v) return fail(CC_ERR_INVALID_ARG, "null %s", name);
    if (!al16(v)) return fail(CC_ERR_INVALID_ARG, "%s not 16-byte aligned", name);
    return CC_OK;
}

extern "C" cc_status cc_launch(cc_plan p, int32_t k, const void* a, const cc_launch_opts* opts,
                               void* stream, int32_t* launches) {
    if (!p || !a) return fail(CC_ERR_INVALID_ARG, "null plan or args");
    if (launches) *launches = 0;
    cc_launch_opts dflt;
    cc_launch_opts_default(&dflt);
    const cc_launch_opts* o = opts ? opts : &dflt;
    if (o->l2_hint < 0 || o->l2_hint > 7) return fail(CC_ERR_INVALID_ARG, "l2_hint %d outside [0, 7]", o->l2_hint);
    if (o->carveout < -1 || o->carveout > 100) return fail(CC_ERR_INVALID_ARG, "carveout %d outside [-1, 100]", o->carveout);
    if (p->device < 0) return fail(CC_ERR_NO_DEVICE, "plan was created host-only");
    int32_t gx = 0, gy = 0;
    CC_TRY(cc_kernel_grid(k, a, &gx, &gy));
    if (gx != p->g.gx || gy != p->g.gy)
        return fail(CC_ERR_INVALID_ARG, "plan grid %dx%d != kernel grid %dx%d", p->g.gx, p->g.gy, gx, gy);
    if (o->backend == CC_BACKEND_TBCLUSTER && k != CC_K_CONV2D)
        return fail(CC_ERR_UNSUPPORTED, "TBCLUSTER backend is implemented for conv2d only");
    DeviceGuard dg;
    CC_TRY(dg.set(p->device));                   // restored on every return path
    cudaStream_t st = (cudaStream_t)stream;
    LaunchCtx c{p, o, st, launches};
    cc_status s = CC_OK;
    switch (k) {
    case CC_K_CENSUS: s = launch_body<CensusBody>(c, CensusParams{0}); break;
    case CC_K_MATVEC: {
        auto* x = (const cc_matvec_args*)a;
        CC_TRY(check_mat(x->A, x->lda, x->m, x->n));
        CC_TRY(check_vec(x->x, x->n, "x")); CC_TRY(check_vec(x->y, x->m, "y"));
        GemvParams gp;
        CC_TRY(gemv_params<32, 32>(&gp, x->A, x->lda, x->m, x->n, x->x, nullptr, x->y, nullptr));
        s = launch_body<MatvecB>(c, gp);
        break;
    }
    case CC_K_ATAX: {
        auto* x = (const cc_atax_args*)a;
        CC_TRY(check_mat(x->A, x->lda, x->m, x->n));
        CC_TRY(check_vec(x->x, x->n, "x")); CC_TRY(check_vec(x->tmp, x->m, "tmp")); CC_TRY(check_vec(x->y, x->n, "y"));
        if (x->m) CC_CUDA(cudaMemsetAsync(x->tmp, 0, sizeof(float) * x->m, st));
        if (x->n) CC_CUDA(cudaMemsetAsync(x->y, 0, sizeof(float) * x->n, st));
        GemvParams g1, g2;
        CC_TRY(gemv_params<32, 256>(&g1, x->A, x->lda, x->m, x->n, x->x, nullptr, x->tmp, nullptr));
        CC_TRY(gemv_params<32, 256>(&g2, x->A, x->lda, x->m, x->n, nullptr, x->tmp, nullptr, x->y));
        s = launch_body<RowB>(c, g1);
        if (s == CC_OK) s = launch_body<ColB>(c, g2);
        break;
    }
    case CC_K_ATAX_FUSED: {
        auto* x = (const cc_atax_args*)a;
        CC_TRY(check_mat(x->A, x->lda, x->m, x->n));
        CC_TRY(check_vec(x->x, x->n, "x")); CC_TRY(check_vec(x->tmp, x->m, "tmp")); CC_TRY(check_vec(x->y, x->n, "y"));
        if (x->n > AtaxFusedBody::kMaxN) return fail(CC_ERR_UNSUPPORTED, "atax_fused: n %d > %d", x->n, AtaxFusedBody::kMaxN);
        if (x->m > 0 && x->n < 1) return fail(CC_ERR_INVALID_ARG, "atax_fused: n < 1");
        if (x->n) CC_CUDA(cudaMemsetAsync(x->y, 0, sizeof(float) * x->n, st));
        s = launch_body<AtaxFusedBody>(c, AtaxFusedParams{x->A, x->lda, x->m, x->n, x->x, x->tmp, x->y});
        break;
    }
    case CC_K_BICG: {
        auto* x = (const cc_bicg_args*)a;
        CC_TRY(check_mat(x->A, x->lda, x->m, x->n));
        CC_TRY(check_vec(x->p, x->n, "p")); CC_TRY(check_vec(x->r, x->m, "r"));
        CC_TRY(check_vec(x->q, x->m, "q")); CC_TRY(check_vec(x->s, x->n, "s"));
        if (x->m) CC_CUDA(cudaMemsetAsync(x->q, 0, sizeof(float) * x->m, st));
        if (x->n) CC_CUDA(cudaMemsetAsync(x->s, 0, sizeof(float) * x->n, st));
        GemvParams gp;
        CC_TRY(gemv_params<32, 256>(&gp, x->A, x->lda, x->m, x->n, x->p, x->r, x->q, x->s));
        s = launch_body<BothB>(c, gp);
        break;
    }
    case CC_K_MVT: {
        auto* x = (const cc_mvt_args*)a;
        CC_TRY(check_mat(x->A, x->lda, x->m, x->n));
        CC_TRY(check_vec(x->y1, x->n, "y1")); CC_TRY(check_vec(x->y2, x->m, "y2"));
        CC_TRY(check_vec(x->x1, x->m, "x1")); CC_TRY(check_vec(x->x2, x->n, "x2"));
        GemvParams gp;
        CC_TRY(gemv_params<32, 256>(&gp, x->A, x->lda, x->m, x->n, x->y1, x->y2, x->x1, x->x2));
        s = launch_body<BothB>(c, gp);
        break;
    }
    case CC_K_JACOBI5: {
        auto* x = (const cc_jacobi5_args*)a;
        CC_TRY(check_mat(x->a, x->ld, x->rows, x->cols));
        CC_TRY(check_mat(x->b, x->ld, x->rows, x->cols));
        if (x->iters < 0) return fail(CC_ERR_INVALID_ARG, "iters < 0");
        const int fuse = x->fuse <= 1 ? 1 : x->fuse;
        if (fuse > 4) return fail(CC_ERR_INVALID_ARG, "jacobi5: fuse %d outside [0, 4]", x->fuse);
        if (fuse > 1 && (x->row_lo != 0 || x->row_hi != 0))
            return fail(CC_ERR_UNSUPPORTED, "jacobi5: fused sweeps with a row window");
        float* src = x->a;
        float* dst = x->b;
        int launches_done = 0;
        // fused launches first (each runs `fuse` sweeps), then single sweeps
        for (int it = 0; fuse > 1 && it + fuse <= x->iters && s == CC_OK; it += fuse) {
            JacobiParams jp;
            memset(&jp, 0, sizeof jp);
            jp.a = src; jp.b = dst; jp.ld = x->ld; jp.rows = x->rows; jp.cols = x->cols;
            jp.row0 = 0; jp.row_end = x->rows;
            if (x->rows > 0 && x->cols > 0) {
                CC_TRY(make_tmap(&jp.tmap, src, x->rows, x->cols, x->ld, ST_COLS, 32 + 2 * fuse));
                CC_TRY(make_tmap(&jp.tmap2, src, x->rows, x->cols, x->ld, ST_COLS2, 32 + 2 * fuse));
            }
            s = fuse == 2 ? launch_body<Jacobi5MultiBody<2>>(c, jp)
              : fuse == 3 ? launch_body<Jacobi5MultiBody<3>>(c, jp)
                          : launch_body<Jacobi5MultiBody<4>>(c, jp);
            std::swap(src, dst);
            ++launches_done;
        }
        const int single = fuse > 1 ? x->iters % fuse : x->iters;
        for (int it = 0; it < single && s == CC_OK; ++it) {
            JacobiParams jp;
            memset(&jp, 0, sizeof jp);
            jp.a = src; jp.b = dst; jp.ld = x->ld; jp.rows = x->rows; jp.cols = x->cols;
            const bool win = x->row_lo != 0 || x->row_hi != 0;
            jp.row0 = win ? x->row_lo : 0;
            jp.row_end = win ? x->row_hi : x->rows;
            if (x->rows > 0 && x->cols > 0) {
                CC_TRY(make_tmap(&jp.tmap, src, x->rows, x->cols, x->ld, ST_COLS, 34));
                CC_TRY(make_tmap(&jp.tmap2, src, x->rows, x->cols, x->ld, ST_COLS2, 34));
                if (o->l2_hint & L2H_HALO_LAST) CC_TRY(make_split(&jp.split, src, x->rows, x->cols, x->ld, 1));
            }
            s = launch_body<Jacobi5Body>(c, jp);
            std::swap(src, dst);
            ++launches_done;
        }
        if (x->result_is_b) *x->result_is_b = (launches_done & 1) ? 1 : 0;
        break;
    }
    case CC_K_JACOBI5_WAVE: {
        auto* x = (const cc_jacobi5_args*)a;
        CC_TRY(check_mat(x->a, x->ld, x->rows, x->cols));
        CC_TRY(check_mat(x->b, x->ld, x->rows, x->cols));
        if (x->iters < 0) return fail(CC_ERR_INVALID_ARG, "iters < 0");
        if (x->row_lo != 0 || x->row_hi != 0) return fail(CC_ERR_UNSUPPORTED, "jacobi5_wave: row window");
        const int K = x->fuse < 1 ? 1 : x->fuse;                  // grid check above bounds it by 8
        const int hl = jw_halo_chunks(K);
        float* src = x->a;
        float* dst = x->b;
        int launches_done = 0;
        for (int it = 0; it < x->iters && s == CC_OK;) {
            const int k = x->iters - it >= K ? K : x->iters - it;  // the tail runs fewer sweeps, same strips
            const JWaveParams jp{src, dst, x->ld, x->rows, x->cols, x->tile_rows == 0 ? JW_ROWS : x->tile_rows};
            s = hl == 1 ? jw_launch<1>(c, jp, k) : jw_launch<2>(c, jp, k);
            std::swap(src, dst);
            ++launches_done;
            it += k;
        }
        if (x->result_is_b) *x->result_is_b = (launches_done & 1) ? 1 : 0;
        break;
    }
    case CC_K_JACOBI5_HALO: {
        auto* x = (const cc_jacobi5_halo_args*)a;
        CC_TRY(check_mat(x->a, x->ld, x->rows, x->cols));
        CC_TRY(check_mat(x->b, x->ld, x->rows, x->cols));
        if (x->iters < 0 || x->sweep0 < 0) return fail(CC_ERR_INVALID_ARG, "iters / sweep0 < 0");
        const bool up = x->up_ll != nullptr, dn = x->dn_ll != nullptr;
        if ((up || dn) && !x->ll) return fail(CC_ERR_INVALID_ARG, "neighbours given but no own ll buffer");
        if (!al16(x->ll) || !al16(x->up_ll) || !al16(x->dn_ll)) return fail(CC_ERR_INVALID_ARG, "ll buffers must be 16-byte aligned");
        if (x->rows - (up ? 1 : 0) - (dn ? 1 : 0) < 1) return fail(CC_ERR_INVALID_ARG, "slab has no owned row");
        float* src = x->a;
        float* dst = x->b;
        for (int it = 0; it < x->iters && s == CC_OK; ++it) {
            JacobiParams jp;
            memset(&jp, 0, sizeof jp);
            jp.a = src; jp.b = dst; jp.ld = x->ld; jp.rows = x->rows; jp.cols = x->cols;
            jp.row0 = 0; jp.row_end = x->rows;
            if (up || dn) {
                jp.h.ll = x->ll; jp.h.up_ll = x->up_ll; jp.h.dn_ll = x->dn_ll;
                jp.h.ldl = (x->cols + 31) & ~31;
                jp.h.sweep = (uint32_t)(x->sweep0 + it + 1);
                jp.h.status = x->status;
            }
            if (x->rows > 0 && x->cols > 0) {
                CC_TRY(make_tmap(&jp.tmap, src, x->rows, x->cols, x->ld, ST_COLS, 34));
                if (o->l2_hint & L2H_HALO_LAST) CC_TRY(make_split(&jp.split, src, x->rows, x->cols, x->ld, 1));
            }
            s = (up || dn) ? launch_body<Jacobi5HaloBody>(c, jp) : launch_body<Jacobi5Body>(c, jp);
            std::swap(src, dst);
        }
        if (x->result_is_b) *x->result_is_b = (x->iters & 1) ? 1 : 0;
        break;
    }
    case CC_K_CONV2D: {
        auto* x = (const cc_conv2d_args*)a;
        CC_TRY(check_mat(x->in, x->ld, x->rows, x->cols));
        CC_TRY(check_mat(x->out, x->ld, x->rows, x->cols));
        if (!x->w) return fail(CC_ERR_INVALID_ARG, "null filter");
        if (x->R == 1) {
            ConvParams<1> cp;
            memset(&cp, 0, sizeof cp);
            cp.in = x->in; cp.out = x->out; cp.ld = x->ld; cp.rows = x->rows; cp.cols = x->cols;
            memcpy(cp.w, x->w, sizeof cp.w);
            if (x->rows > 0 && x->cols > 0) {
                CC_TRY(make_tmap(&cp.tmap, x->in, x->rows, x->cols, x->ld, ST_COLS, 34));
                CC_TRY(make_tmap(&cp.tmap2, x->in, x->rows, x->cols, x->ld, ST_COLS2, 34));
                if (o->l2_hint & L2H_HALO_LAST) CC_TRY(make_split(&cp.split, x->in, x->rows, x->cols, x->ld, 1));
            }
            s = o->backend == CC_BACKEND_TBCLUSTER ? launch_tbc<1>(c, cp)
                                                   : launch_body<Conv2dBody<1>>(c, cp);
        } else if (x->R == 3) {
            ConvParams<3> cp;
            memset(&cp, 0, sizeof cp);
            cp.in = x->in; cp.out = x->out; cp.ld = x->ld; cp.rows = x->rows; cp.cols = x->cols;
            memcpy(cp.w, x->w, sizeof cp.w);
            if (x->rows > 0 && x->cols > 0) {
                CC_TRY(make_tmap(&cp.tmap, x->in, x->rows, x->cols, x->ld, ST_COLS, 38));
                CC_TRY(make_tmap(&cp.tmap2, x->in, x->rows, x->cols, x->ld, ST_COLS2, 38));
                if (o->l2_hint & L2H_HALO_LAST) CC_TRY(make_split(&cp.split, x->in, x->rows, x->cols, x->ld, 3));
            }
            s = o->backend == CC_BACKEND_TBCLUSTER ? launch_tbc<3>(c, cp)
                                                   : launch_body<Conv2dBody<3>>(c, cp);
        } else {
            return fail(CC_ERR_UNSUPPORTED, "conv2d radius %d (1 or 3 supported)", x->R);
        }
        break;
    }
    case CC_K_SPMV: case CC_K_SPMV_SHUB: {
        auto* x = (const cc_spmv_args*)a;
        if (x->rows < 0 || x->cols < 0 || x->nnz < 0 || x->nnz > INT32_MAX) return fail(CC_ERR_INVALID_ARG, "spmv sizes");
        if (!x->row_ptr || !x->part || !x->y || (x->nnz && (!x->col || !x->val || !x->x)))
            return fail(CC_ERR_INVALID_ARG, "spmv null pointer");
        if (x->n_hot < 0 || (x->n_hot > 0 && (!x->hot || !x->xh)))
            return fail(CC_ERR_INVALID_ARG, "spmv hub-column form: n_hot %d, hot/xh required", x->n_hot);
        if (k == CC_K_SPMV_SHUB) {
            if (o->backend != CC_BACKEND_AGENT && o->backend != CC_BACKEND_AGENT_IDENTITY &&
                o->backend != CC_BACKEND_AGENT_STATIC)
                return fail(CC_ERR_UNSUPPORTED, "spmv_shub: persistent backends only (agent / identity / static)");
            if (x->n_hot > 0 && !al16(x->xh)) return fail(CC_ERR_INVALID_ARG, "spmv_shub: xh must be 16-byte aligned");
        }
        if (x->rows) CC_CUDA(cudaMemsetAsync(x->y, 0, sizeof(float) * x->rows, st));
        if (x->n_hot > 0) {
            k_spmv_hot_gather<<<std::min(148 * 4, (x->n_hot + 255) / 256), 256, 0, st>>>(x->x, x->hot, x->xh, x->n_hot);
            cudaError_t e = cudaGetLastError();
            if (e != cudaSuccess) return cuda_fail(e, "spmv hub gather");
            if (launches) ++*launches;
        }
        const SpmvParams sp{x->rows, x->nnz, x->row_ptr, x->col, x->val, x->x, x->y, x->part,
                            x->n_hot > 0 ? x->xh + x->n_hot : nullptr, x->n_hot};
        s = k == CC_K_SPMV_SHUB ? launch_body<SpmvShubBody>(c, sp) : launch_body<SpmvBody>(c, sp);
        break;
    }
    case CC_K_HIST64: {
        auto* x = (const cc_hist64_args*)a;
        if (!x->counts || (x->n > 0 && !x->data)) return fail(CC_ERR_INVALID_ARG, "hist64 null pointer");
        if (x->n > 0 && !al16(x->data)) return fail(CC_ERR_INVALID_ARG, "hist64: data must be 16-byte aligned");
        CC_CUDA(cudaMemsetAsync(x->counts, 0, 64 * sizeof(uint32_t), st));
        s = launch_body<HistBody>(c, HistParams{x->data, x->n, x->counts});
        break;
    }
    default:
        s = fail(CC_ERR_INVALID_ARG, "unknown kernel %d", k);
    }
    return s;
}

extern "C" cc_status cc_l1_reuse_probe(int32_t ctas, int32_t stagger_cycles, const float* input, int32_t* smid,
                                     uint32_t* ticks, float* sink, void* stream) {
    if (ctas < 0 || stagger_cycles < 0) return fail(CC_ERR_INVALID_ARG, "ctas %d / stagger %d", ctas, stagger_cycles);
    if (ctas == 0) return CC_OK;
    if (!input || !smid || !ticks || !sink) return fail(CC_ERR_INVALID_ARG, "l1 reuse probe: null pointer");
    k_l1_reuse_probe<<<ctas, 32, 0, (cudaStream_t)stream>>>(input, smid, ticks, sink, stagger_cycles);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "l1 reuse probe");
    return CC_OK;
}

// ---- peer memory for the fused halo (S§8(f)4) -------------------------------
extern "C" cc_status cc_peer_access(int32_t device, int32_t peer) {
    if (device < 0 || peer < 0) return fail(CC_ERR_INVALID_ARG, "device %d / peer %d", device, peer);
    if (device == peer) return CC_OK;
    int ok = 0;
    CC_CUDA(cudaDeviceCanAccessPeer(&ok, device, peer));
    if (!ok) return fail(CC_ERR_UNSUPPORTED, "device %d cannot access peer %d", device, peer);
    int prev = 0;
    CC_CUDA(cudaGetDevice(&prev));
    CC_CUDA(cudaSetDevice(device));
    cudaError_t e = cudaDeviceEnablePeerAccess(peer, 0);
    cudaSetDevice(prev);
    if (e == cudaErrorPeerAccessAlreadyEnabled) { cudaGetLastError(); return CC_OK; }
    if (e != cudaSuccess) return cuda_fail(e, "cudaDeviceEnablePeerAccess");
    return CC_OK;
}
extern "C" cc_status cc_l2_persist(void* stream, const void* ptr, size_t bytes, float hit_ratio) {
    cudaStream_t st = (cudaStream_t)stream;
    cudaStreamAttrValue v;
    memset(&v, 0, sizeof v);
    if (bytes == 0) {
        v.accessPolicyWindow.num_bytes = 0;
        CC_CUDA(cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &v));
        CC_CUDA(cudaCtxResetPersistingL2Cache());
        return CC_OK;
    }
    if (!ptr || !(hit_ratio > 0.f && hit_ratio <= 1.f)) return fail(CC_ERR_INVALID_ARG, "l2 persist: ptr / hit_ratio");
    int dev = 0, max_persist = 0, max_window = 0;
    CC_CUDA(cudaGetDevice(&dev));
    CC_CUDA(cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, dev));
    CC_CUDA(cudaDeviceGetAttribute(&max_window, cudaDevAttrMaxAccessPolicyWindowSize, dev));
    const size_t win = std::min(bytes, (size_t)max_window);
    CC_CUDA(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, std::min(win, (size_t)max_persist)));
    v.accessPolicyWindow.base_ptr = const_cast<void*>(ptr);
    v.accessPolicyWindow.num_bytes = win;
    v.accessPolicyWindow.hitRatio = hit_ratio;
    v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    CC_CUDA(cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &v));
    return CC_OK;
}

// IPC maps whole allocations: the handle names the allocation holding dptr
// (a caching allocator hands out sub-blocks), *offset is dptr's byte offset in it.
extern "C" cc_status cc_ipc_handle(const void* dptr, void* handle64, uint64_t* offset) {
    if (!dptr || !handle64 || !offset) return fail(CC_ERR_INVALID_ARG, "null pointer");
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle size");
    using RangeFn = CUresult (*)(CUdeviceptr*, size_t*, CUdeviceptr);
    static RangeFn range = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        cudaDriverEntryPointQueryResult q;
        void* f = nullptr;
        if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            range = (RangeFn)f;
    });
    if (!range) return fail(CC_ERR_UNSUPPORTED, "cuMemGetAddressRange unavailable");
    CUdeviceptr base = 0;
    size_t size = 0;
    CUresult r = range(&base, &size, (CUdeviceptr)dptr);
    if (r != CUDA_SUCCESS) return fail(CC_ERR_CUDA, "cuMemGetAddressRange failed (%d)", (int)r);
    cudaIpcMemHandle_t h;
    CC_CUDA(cudaIpcGetMemHandle(&h, (void*)base));
    memcpy(handle64, &h, 64);
    *offset = (uint64_t)((CUdeviceptr)dptr - base);
    return CC_OK;
}
extern "C" cc_status cc_ipc_open(const void* handle64, int32_t device, void** dptr) {
    if (!handle64 || !dptr || device < 0) return fail(CC_ERR_INVALID_ARG, "null pointer / device");
    cudaIpcMemHandle_t h;
    memcpy(&h, handle64, 64);
    int prev = 0;
    CC_CUDA(cudaGetDevice(&prev));
    CC_CUDA(cudaSetDevice(device));
    cudaError_t e = cudaIpcOpenMemHandle(dptr, h, cudaIpcMemLazyEnablePeerAccess);
    cudaSetDevice(prev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaIpcOpenMemHandle");
    return CC_OK;
}
extern "C" cc_status cc_ipc_close(void* dptr) {
    if (!dptr) return fail(CC_ERR_INVALID_ARG, "null pointer");
    CC_CUDA(cudaIpcCloseMemHandle(dptr));
    return CC_OK;
}

extern "C" cc_status cc_spmv_partition(const cc_spmv_args* x, int32_t* part, void* stream) {
    if (!x || !part || !x->row_ptr) return fail(CC_ERR_INVALID_ARG, "null argument");
    int32_t gx = 0, gy = 0;
    CC_TRY(cc_kernel_grid(CC_K_SPMV, x, &gx, &gy));
    int n = gx + 1;
    k_spmv_partition<<<(n + 255) / 256, 256, 0, (cudaStream_t)stream>>>(x->row_ptr, x->rows, x->nnz, gx, part);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "spmv partition");
    return CC_OK;
}

extern "C" cc_status cc_spmv_inspect(const cc_spmv_args* x, int32_t max_hot, int32_t* hot, int32_t* col_hot,
                                     int32_t* scratch, int32_t* n_hot, void* stream) {
    if (!x || !n_hot || !scratch || max_hot < 0 || (x->nnz && (!x->col || !col_hot)) || (max_hot && !hot))
        return fail(CC_ERR_INVALID_ARG, "spmv inspect: null argument or max_hot < 0");
    if (x->cols < 0 || x->nnz < 0 || x->nnz > INT32_MAX) return fail(CC_ERR_INVALID_ARG, "spmv inspect: sizes");
    *n_hot = 0;
    cudaStream_t st = (cudaStream_t)stream;
    const int32_t cols = x->cols;
    int32_t* deg = scratch;
    int32_t* hist = scratch + cols;
    const int grid = 148 * 8;
    CC_CUDA(cudaMemsetAsync(scratch, 0, sizeof(int32_t) * ((size_t)cols + 65536 + 2), st));
    if (x->nnz) k_spmv_col_degree<<<grid, 256, 0, st>>>(x->col, x->nnz, deg);
    if (cols) k_spmv_deg_hist<<<grid, 256, 0, st>>>(deg, cols, hist);
    std::vector<int32_t> h(65536);
    CC_CUDA(cudaMemcpyAsync(h.data(), hist, sizeof(int32_t) * 65536, cudaMemcpyDeviceToHost, st));
    CC_CUDA(cudaStreamSynchronize(st));
    // degree-sorted view of the histogram: G(d) = #columns of degree > d; the
    // k-th most referenced column (k >= 1) has the degree d with
    // G(d) < k <= G(d) + h[d].  Unreferenced columns are never hubs.
    int64_t referenced = 0;
    for (int32_t d = 1; d < 65536; ++d) referenced += h[d];
    const int32_t used = (int32_t)std::min<int64_t>(referenced, max_hot);
    const int32_t T = std::min(used, (int32_t)CC_SPMV_SHUB_SLOTS);
    auto kth = [&](int64_t k, int64_t* above) {   // degree of the k-th, and G(that degree)
        int64_t g = 0;
        for (int32_t d = 65535; d >= 1; --d) {
            if (g + h[d] >= k) { *above = g; return d; }
            g += h[d];
        }
        *above = g;
        return 1;
    };
    int64_t n_a = 0, g_b = 0;
    const int32_t dA = T > 0 ? kth(T, &n_a) : 65536;
    const int32_t dB = used > 0 ? kth(used, &g_b) : 65536;
    const int32_t n_b = dA > dB ? (int32_t)(g_b - T) : 0;
    int32_t* ctr = hist;                            // the histogram is on the host now: its first words count
    CC_CUDA(cudaMemsetAsync(ctr, 0, 4 * sizeof(int32_t), st));
    k_spmv_hot_assign<<<grid, 256, 0, st>>>(deg, cols, dA, (int32_t)n_a, T, dB, n_b, used, ctr, hot);
    if (x->nnz) k_spmv_col_encode<<<grid, 256, 0, st>>>(x->col, x->nnz, deg, col_hot);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "spmv inspect");
    CC_CUDA(cudaStreamSynchronize(st));
    *n_hot = used;
    return CC_OK;
}

extern "C" const char* cc_status_string(cc_status s) {
    switch (s) {
    case CC_OK: return "ok";
    case CC_ERR_INVALID_ARG: return "invalid argument";
    case CC_ERR_OVERFLOW: return "size overflow";
    case CC_ERR_NOT_PERMUTATION: return "user order is not a permutation";
    case CC_ERR_CUDA: return "CUDA error";
    case CC_ERR_NCCL: return "NCCL error";
    case CC_ERR_UNSUPPORTED: return "unsupported";
    case CC_ERR_NO_DEVICE: return "plan has no device";
    case CC_ERR_BUSY: return "plan workspace busy on another stream";
    }
    return "unknown status";
}
extern "C" const char* cc_last_error(void) { return g_err.c_str(); }
extern "C" int cc_last_cuda_error(void) { return g_cuda_err; }
extern "C" const char* cc_version(void) { return "libctaclust 0.1 (sm_100a)"; }
