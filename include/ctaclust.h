/*
 * ctaclust.h -- C ABI of libctaclust, a B200 (sm_100a) implementation of
 * locality-aware CTA clustering (Li, Song, Liu, Liu, Kumar, Corporaal,
 * "Locality-Aware CTA Clustering for Modern GPUs", ASPLOS'17).
 * Citations "P:<n>" are line numbers of the paper transcript;
 * the section / equation / listing is named next to each.
 *
 * Conventions (all entry points):
 *  - Every function returns cc_status (CC_OK == 0).  Nothing aborts, throws or
 *    prints across the ABI; cc_last_error() gives a thread-local message for the
 *    most recent failure on the calling thread.
 *  - Pointers are plain host or device pointers as stated per argument; no
 *    framework types.  The caller owns every buffer it passes; the library owns
 *    only what a cc_plan holds (its device tables and default workspace).
 *  - Launches are asynchronous on the caller's stream (a cudaStream_t passed as
 *    void*; NULL = legacy default stream).  Errors detected at launch time are
 *    returned; asynchronous kernel faults surface at the caller's next
 *    synchronisation as usual for CUDA.
 *  - Sizes are validated; logical grids whose CTA count overflows int32 give
 *    CC_ERR_OVERFLOW.
 */
#ifndef CTACLUST_H
#define CTACLUST_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    CC_OK = 0,
    CC_ERR_INVALID_ARG = -1,     /* null/negative/misaligned argument, grid mismatch */
    CC_ERR_OVERFLOW = -2,        /* gx*gy (or a derived size) exceeds int32 */
    CC_ERR_NOT_PERMUTATION = -3, /* USER order is not a permutation of [0, gx*gy) */
    CC_ERR_CUDA = -4,            /* a CUDA runtime call failed; see cc_last_cuda_error() */
    CC_ERR_NCCL = -5,            /* reserved for the NCCL-backed entry points */
    CC_ERR_UNSUPPORTED = -6,     /* valid request this build / device cannot serve */
    CC_ERR_NO_DEVICE = -7,       /* plan created host-only (device < 0) was asked to launch */
    CC_ERR_BUSY = -8             /* reserved (round 1 refused an agent launch on another
                                    stream while the plan's workspace was in use; cc_launch
                                    now orders such a launch after the previous one) */
} cc_status;

/* ---------------------------------------------------------------------------
 * Planner: Step 1 partitioning f and Step 2 inverting f^-1 (§4.2)
 *
 * The logical grid O of gx*gy CTAs is put in the order of a CTA indexing method
 * (Fig. 7) and cut into M balanced contiguous clusters (Eq. 2-5,
 * P:1869-1875): with q = |V|/M and r = |V|%M the first r clusters hold q+1 CTAs,
 * the rest q (readings R1/R2 for the garbled Eq. 4/5).  v denotes a
 * CTA's position in that order; slot (w, i) is position w of cluster i and
 * v = f^-1(w, i) = i*(q+1) + w + min(r-i, 0)   (Eq. 7).
 * Tables name CTAs by their row-major linear id lin = by*gx + bx.
 * ------------------------------------------------------------------------- */
typedef enum {
    CC_ORDER_ROW = 0,  /* v = by*gx + bx : the paper's "Y-partitioning"   */
    CC_ORDER_COL = 1,  /* v = bx*gy + by : the paper's "X-partitioning"   */
    CC_ORDER_TILE = 2, /* tile_w x tile_h CTA tiles, row-major over tiles and inside
                          each tile, edge tiles clipped (Fig. 7 tile panel; R6)    */
    CC_ORDER_USER = 3  /* arbitrary order: user_order[v] = lin ("customized") */
} cc_order;

typedef struct {
    int32_t gx, gy;             /* logical grid (gridDim.x, gridDim.y of O); >= 0    */
    int32_t order;              /* cc_order                                         */
    int32_t tile_w, tile_h;     /* TILE only, >= 1                                  */
    int32_t num_clusters;       /* M; 0 => number of SMs of `device` ("size
                                   of C equal to the number of SMs, 1-to-1")        */
    const int32_t* user_order;  /* HOST, gx*gy entries, USER only; copied at create  */
    int32_t device;             /* CUDA ordinal owning the device tables; -1 => a
                                   host-only plan (tables/lookups, no launches)     */
} cc_plan_desc;

typedef struct cc_plan_s* cc_plan;   /* opaque; immutable after create except for
                                        its self-resetting launch workspace        */

/* Build the partition.  Errors: INVALID_ARG (null, negative grid, M < 1 when
 * device < 0, bad tile dims, bad order), OVERFLOW, NOT_PERMUTATION, CUDA. */
cc_status cc_plan_create(const cc_plan_desc* desc, cc_plan* out);
/* Free the plan.  The caller must have synchronised every stream that used it. */
cc_status cc_plan_destroy(cc_plan plan);
/* |V|, M, q = |V|/M, r = |V|%M.  Any output pointer may be NULL. */
cc_status cc_plan_info(cc_plan plan, int64_t* num_ctas, int32_t* num_clusters,
                       int32_t* q, int32_t* r);
/* Copy the partition to HOST arrays the caller allocated: perm[|V|] (cluster-
 * major list of lin ids: perm[offsets[i] + w] = lin of slot (w,i)) and
 * offsets[M+1].  Either pointer may be NULL. */
cc_status cc_plan_table(cc_plan plan, int32_t* perm, int32_t* offsets);
/* f(v) = (w, i)  (Eq. 2-5).  INVALID_ARG when v is outside [0, |V|). */
cc_status cc_plan_lookup(cc_plan plan, int32_t v, int32_t* w, int32_t* i);
/* f^-1(w, i) = v (Eq. 7).  INVALID_ARG when (w, i) is not a slot of the plan. */
cc_status cc_plan_invert(cc_plan plan, int32_t w, int32_t i, int32_t* v);

/* ---------------------------------------------------------------------------
 * Device facts used for binding (§4.2.3 Step 3)
 * ------------------------------------------------------------------------- */
/* num_sms = cudaDevAttrMultiProcessorCount; smid_span = %nsmid (the range of the
 * virtual %smid register); l2_bytes = L2 size.  Outputs may be NULL. */
cc_status cc_device_info(int32_t device, int32_t* num_sms, int32_t* smid_span,
                         int32_t* l2_bytes);
/* The dense SM rank table the agent runtime binds clusters with: rank_of_smid
 * (HOST, smid_span entries) maps a %smid value to a rank in [0, num_sms) or -1
 * if that smid was never observed.  Built once per device by a probe kernel
 * (reading R7: %smid is virtual and may be sparse, so cluster i binds to the
 * SM of dense rank i rather than to smid i as Listing 5 l.14-15 does). */
cc_status cc_sm_rank_table(int32_t device, int32_t* rank_of_smid, int32_t capacity,
                           int32_t* smid_span);

/* ---------------------------------------------------------------------------
 * Launch: Step 3 binding + the task loop (§4.2.3-4.3, Listing 5)
 * ------------------------------------------------------------------------- */
typedef enum {
    CC_BACKEND_DEFAULT = 0,        /* hardware CTA order: grid (gx, gy), body(blockIdx) --
                                      the paper's baseline "BSL"              */
    CC_BACKEND_AGENT = 1,          /* agent-based clustering (Listing 5; "CLU",
                                      with throttling "CLU+TOT")                       */
    CC_BACKEND_TBCLUSTER = 2,      /* Blackwell thread-block clusters: the hardware form
                                      of clustering (conv2d only in this build): a
                                      persistent grid of clusters of cluster_size CTAs
                                      on vertically adjacent tiles; the rows a CTA pair
                                      shares are fetched once and TMA-multicast to both */
    CC_BACKEND_AGENT_IDENTITY = 3, /* persistence-only control: same agents, one global
                                      queue in row-major order, no locality grouping   */
    CC_BACKEND_REDIRECT = 4,       /* redirection-based clustering "RD" (Listing 4,
                                      Eq. 8 + Eq. 7; relies on RR dispatch)    */
    CC_BACKEND_AGENT_STATIC = 5    /* static binding: grid = the plan's M CTAs, CTA i runs
                                      cluster i's tasks in Eq. 7 order through the same
                                      staging ring.  A cluster's tasks share an SM by
                                      construction (one CTA), with no %smid probe, queue
                                      atomics, stealing or workspace; active_agents and
                                      steal are ignored.  Pick M (num_clusters) as a
                                      multiple of the SM count x resident CTAs.      */
} cc_backend;

typedef enum { CC_STAGING_DEFAULT = 0, CC_STAGING_TMA = 1, CC_STAGING_L1 = 2, CC_STAGING_DIRECT = 3 } cc_staging;

/* L2 eviction-priority hints (S§8(f)2: the paper's bypassing of streaming
 * accesses, §4.3(II), carried to B200's L2 with createpolicy +
 * .L2::cache_hint).  Bits: 1 = the kernel's streamed operand is evict_first
 * (gemv: A; stencils: the output; SpMV: col/val); 2 = its reused operand is
 * evict_last (gemv: the vector slices; stencils: the TMA-staged input with
 * its halo; SpMV: x); 4 = stencils (Jacobi, conv) only: stage each tile as two
 * TMA boxes, the rows the next tile row re-reads as its top halo evict_last
 * and the rest of the input evict_first (takes precedence over bit 2 there;
 * ignored by the other kernels).  0 = no hint (default).  One-shot backends
 * (default, redirect) ignore every bit. */
typedef enum { CC_L2_HINT_NONE = 0, CC_L2_HINT_STREAM_FIRST = 1, CC_L2_HINT_REUSE_LAST = 2,
               CC_L2_HINT_BOTH = 3, CC_L2_HINT_HALO_LAST = 4 } cc_l2_hint;

typedef struct {
    int32_t backend;        /* cc_backend                                               */
    int32_t active_agents;  /* agents per SM that work (throttling, §4.3(I));
                               0 => max_agents                                          */
    int32_t max_agents;     /* agents launched per SM (MAX_AGENTS, Fig. 10); 0 => the
                               occupancy limit of the kernel                            */
    int32_t stages;         /* agent backends: depth of the per-agent shared-memory ring
                               the scheduler warp stages upcoming tasks into -- the
                               B200 form of "prefetch the next CTA" (§4.3(III),
                               Listing 5 l.34-37); 0 => the kernel's default, 1..8;
                               rounded up to a multiple of the body's consumer
                               groups (each ring slot belongs to one group)          */
    int32_t batch;          /* logical CTAs claimed per queue atomic; 0 => default   */
    int32_t staging;        /* how a task's input tile reaches the body (cc_staging):
                               0 default (= TMA), 1 TMA: one 2D tensor load per tile,
                               L2 -> smem, L1 bypassed (the B200 form of "BPS",
                               §4.3(II)); 2 cp.async.ca: 16-byte copies
                               that also allocate in L1, so neighbouring tasks on the
                               same SM hit the shared halo (the paper's L1 reuse;
                               stencils only); 3 direct: no producer staging, the
                               consumers load through L1 themselves (the plain
                               kernel form).  SpMV always loads directly.            */
    int32_t steal;          /* 1 (default) => an agent whose cluster queue is empty
                               takes work from other clusters, so every CTA runs exactly
                               once whatever the hardware does with agent placement
                               (reading R10); 0 => paper-faithful: CTAs of a cluster
                               with no active agent are NOT run (census shows it)       */
    int32_t cluster_size;   /* TBCLUSTER: CTAs per cluster along y (1, 2, 4 or 8)       */
    uint32_t* d_census;     /* DEVICE, |V|, optional: census[lin] += 1 per execution;
                               caller zeroes it                                        */
    int32_t* d_exec_sm;     /* DEVICE, |V|, optional: %smid that executed lin          */
    int32_t* d_map;         /* DEVICE, |V|, optional: d_map[v] = lin executed for the
                               slot at order position v (agent/redirect/identity)      */
    int32_t l2_hint;        /* cc_l2_hint bits (0..7); default 0                        */
    int32_t carveout;       /* preferred shared-memory carveout of the launched kernel,
                               percent of the SM's L1/shared array (0..100; the rest
                               is L1), set with cudaFuncAttributePreferredShared-
                               MemoryCarveout before the launch; -1 (default) = the
                               driver's choice.  Agents per SM are recomputed under it. */
} cc_launch_opts;

/* Fill *opts with defaults: AGENT backend, max/active from occupancy, steal = 1,
 * stages/batch per kernel, cluster_size = 2, no census/map, no L2 hint,
 * carveout -1. */
cc_status cc_launch_opts_default(cc_launch_opts* opts);

typedef enum {
    CC_K_CENSUS = 0,   /* empty body: exercises binding/census only                */
    CC_K_MATVEC = 1,   /* cc_matvec_args   (Listing 2; config 1)           */
    CC_K_ATAX = 2,     /* cc_atax_args     (Table 2 ATX; config 2)                  */
    CC_K_BICG = 3,     /* cc_bicg_args     (Table 2 BC)                             */
    CC_K_MVT = 4,      /* cc_mvt_args      (Table 2 MVT)                            */
    CC_K_JACOBI5 = 5,  /* cc_jacobi5_args  (config 3)                               */
    CC_K_CONV2D = 6,   /* cc_conv2d_args   (config 4)                               */
    CC_K_SPMV = 7,     /* cc_spmv_args     (config 5)                               */
    CC_K_HIST64 = 8,   /* cc_hist64_args   (S§8(f)3, the paper's HST)               */
    CC_K_JACOBI5_HALO = 9, /* cc_jacobi5_halo_args (S§8(f)4: sharded sweep, fused peer halo) */
    CC_K_ATAX_FUSED = 10, /* cc_atax_args: one-pass ATAX (both PolyBench kernels per row) */
    CC_K_SPMV_SHUB = 11,  /* cc_spmv_args: SpMV with the hub array in each agent's shared memory */
    CC_K_JACOBI5_WAVE = 12 /* cc_jacobi5_args: fused sweeps as strip wavefronts carried across tiles (R34) */
} cc_kernel;

/* CC_K_CENSUS: no data. */
typedef struct { int32_t gx, gy; } cc_census_args;

/* y += A x, A m x n row-major fp32 (DEVICE), lda % 4 == 0, lda >= n, A/x/y
 * 16-byte aligned.  Logical CTA (bx, by) = 32 x 32 tile: rows 32*by.., columns
 * 32*bx.. (Listing 2 layout: bx -> B[idx], by -> C[idy]); grid ceil(n/32) x
 * ceil(m/32).  y is NOT zeroed (Listing 2 accumulates with atomicAdd). */
typedef struct { const float* A; int64_t lda; int32_t m, n; const float* x; float* y; } cc_matvec_args;

/* The ATAX/BICG/MVT family share one tile body: logical CTA (bx, by) is the
 * 32 x 256 tile A[32*by .. +32, 256*bx .. +256]; grid ceil(n/256) x ceil(m/32).
 * A m x n row-major fp32 DEVICE, lda % 4 == 0, lda >= n, 16-byte aligned. */
/* ATAX: tmp = A x ; y = A^T tmp (two launches; tmp and y are zeroed by the call). */
typedef struct { const float* A; int64_t lda; int32_t m, n; const float* x; float* tmp; float* y; } cc_atax_args;
/* CC_K_ATAX_FUSED: the same ATAX (tmp = A x, y = A^T tmp; tmp and y written /
 * zeroed by the call) over ONE read of A (Table 2 ATX; reading R31):
 * logical CTA (0, i) is row i; the agent owning it computes tmp[i] and adds
 * A[i][:] * tmp[i] into its register-held y partial while the row sits in its
 * shared-memory ring (x held in registers), flushing y once per agent with
 * vector REDs.  Grid 1 x m.  1 <= n <= 16384; A rows 16-byte aligned (lda % 4
 * == 0).  Meant for the persistent backends (agent / identity / static): a
 * one-shot CTA flushes n REDs per row.  Errors: INVALID_ARG, UNSUPPORTED
 * (n > 16384, TBCLUSTER). */
/* BICG: q = A p ; s = A^T r (one fused pass; q and s zeroed by the call). */
typedef struct { const float* A; int64_t lda; int32_t m, n; const float* p; const float* r; float* q; float* s; } cc_bicg_args;
/* MVT: x1 += A y1 ; x2 += A^T y2 (one fused pass, in place). */
typedef struct { const float* A; int64_t lda; int32_t m, n; const float* y1; const float* y2; float* x1; float* x2; } cc_mvt_args;

/* 5-point Jacobi sweeps (R14, PolyBench jacobi-2d): b[i][j] =
 * 0.2f*((((c + w) + e) + s) + n) in fp32 on the interior (s = row i+1,
 * n = row i-1), boundary rows/cols copied.  `iters` sweeps ping-pong
 * a -> b -> a ...; on return *result_is_b (HOST, optional) says which buffer
 * holds the last sweep.  rows x cols fp32 DEVICE with leading dim ld (% 4 == 0).
 * Row window (for the slab-sharded driver's boundary / interior split,
 * S§8(e)): when row_hi > row_lo only output rows [row_lo, row_hi) of b are
 * written (rows outside it are left untouched; every input row is still
 * read as in the full sweep); 0 <= row_lo < row_hi <= rows.  row_lo = row_hi
 * = 0: all rows.  Logical CTA = 32 x 32 output tile of the window; grid
 * ceil(cols/32) x ceil((row_hi - row_lo)/32) (ceil(rows/32) without a window). */
typedef struct { float* a; float* b; int64_t ld; int32_t rows, cols; int32_t iters; int32_t* result_is_b;
                 int32_t row_lo, row_hi;
                 int32_t fuse;   /* sweeps per launch (reading R32): 0 or 1 = one; 2, 3 or 4 = that many
                                    consecutive sweeps per launch (each tile staged once with a fuse-row
                                    halo, the intermediate sweeps recomputed on chip), bit-identical to
                                    single sweeps; iters % fuse remaining sweeps run one per launch.
                                    Not with a row window (UNSUPPORTED). */
                 int32_t tile_rows; /* CC_K_JACOBI5_WAVE only: logical CTA height in rows, 0 = 64; 8..1024
                                    (INVALID_ARG otherwise).  Small tiles favour the carried COL clusters,
                                    tall ones hardware order; ignored by CC_K_JACOBI5. */
               } cc_jacobi5_args;

/* CC_K_JACOBI5_WAVE -- the same sweeps (CC_K_JACOBI5's arithmetic, bit-identical,
 * `iters` sweeps ping-ponging a -> b -> a, *result_is_b as there) run K = fuse
 * (1..8; 0 = 1) at a time by warp agents streaming column strips
 * (reading R34, §4.2 P:1793 / Listing 5).  Logical CTA
 * (bx, by) = output rows [T by, T by + T) x columns [WS bx, WS bx + WS),
 * T = tile_rows (default 64), WS = 120 for K <= 4 and 112 for K = 5..8; grid
 * ceil(cols/WS) x ceil(rows/T).  One launch runs K sweeps: a warp ingests its
 * tile's input rows from T by - K to T by + T + K and keeps every intermediate sweep's last two rows in
 * registers; when its next logical CTA is the tile directly below (the next
 * position of a COL-ordered cluster) it carries them over instead of re-reading
 * and re-sweeping the 2K-row overlap.  The tail launch runs iters % K sweeps
 * on the same grid.  Backends: DEFAULT (one warp per logical CTA, hardware
 * order); AGENT and AGENT_IDENTITY (agents = worker warps: 24 (fuse <= 3),
 * 20 (fuse 4) or 15 in one CTA per SM beside a scheduler warp that pops their
 * logical CTAs; max_agents / active_agents count workers per SM; batch > 0 =
 * tiles per queue claim, 0 = chunked claims: 3/4 of a queue in one contiguous
 * chunk per agent, the rest tile by tile); AGENT_STATIC (worker i runs
 * cluster i: ceil(M / workers) CTAs).  The L2 hint and staging options are
 * ignored.  No row window (UNSUPPORTED); TBCLUSTER / REDIRECT UNSUPPORTED;
 * fuse outside [0, 8] INVALID_ARG. */

/* CC_K_JACOBI5_HALO -- S§8(f)4: one rank's slab of the slab-sharded Jacobi
 * (S§8(e), config 3) with the per-sweep halo exchange fused into the sweep
 * kernel over peer memory, replacing cc_halo_exchange's NCCL send/recv.
 * The slab a/b (DEVICE, rows x cols, ld) holds this rank's owned rows plus one
 * halo row above (row 0, when up_ll != NULL) and below (row rows-1, when
 * dn_ll != NULL); the arithmetic is CC_K_JACOBI5's (halo and global boundary
 * rows are fixed during a sweep).  Halo values cross as 64-bit words {fp32
 * bits, absolute sweep number} ("LL" form, no fences): in sweep s the threads
 * computing the first (last) owned row also store it, tagged s, into the
 * upper (lower) neighbour's LL buffer of parity s & 1; in sweep s > 1 the
 * tiles needing a halo row read this rank's LL buffer of parity (s-1) & 1 (a
 * bulk copy riding with the tile's TMA) and re-poll any word not yet carrying
 * tag s-1.  Sweep 1 uses the halo rows already in a.  The body visits the
 * boundary tile rows first (a fixed bijection on tile rows).
 *   a, b            this call's first source / destination (ping-pong as in
 *                   CC_K_JACOBI5; *result_is_b as there)
 *   iters, sweep0   runs absolute sweeps sweep0+1 .. sweep0+iters
 *   ll              DEVICE uint64[4 * ldl], ldl = cols rounded up to 32, 16-byte
 *                   aligned: [parity 0/1][side 0 = from up / 1 = from down][ldl];
 *                   zeroed by the caller (on every rank, before any rank's
 *                   sweep 1) when sweep0 = 0
 *   up_ll, dn_ll    the neighbours' `ll`, mapped into this process (same
 *                   device, cc_peer_access, or cc_ipc_open); NULL = no such
 *                   neighbour (that slab edge is the global boundary)
 *   status          DEVICE int32, optional: set to 1 if a poll exceeded 4 s in
 *                   total (a neighbour not running); results are then invalid
 * Every rank uses the same cols.  Halo rows of b are not written.  Launches of
 * neighbouring ranks may run concurrently (one GPU each) or be interleaved
 * sweep by sweep on one stream (virtual slabs on one GPU); a rank's sweep s
 * must not be queued behind a neighbour's sweep s+1 on one stream.
 * Errors: INVALID_ARG (sizes, a neighbour without `ll`, misaligned ll, owned
 * rows < 1), UNSUPPORTED (TBCLUSTER backend). */
typedef struct {
    float* a; float* b; int64_t ld; int32_t rows, cols; int32_t iters; int32_t sweep0; int32_t* result_is_b;
    uint64_t* ll; uint64_t* up_ll; uint64_t* dn_ll;
    int32_t* status;
} cc_jacobi5_halo_args;

/* Peer memory for CC_K_JACOBI5_HALO (S§8(f)4).  cc_peer_access enables P2P
 * loads/stores from `device` to `peer` (NVLink on a B200 box); a no-op when
 * device == peer or access is already enabled.  cc_ipc_handle exports the
 * DEVICE allocation holding dptr (cudaIpcGetMemHandle; 64-byte HOST handle
 * out) and dptr's byte offset in it (*offset, HOST); cc_ipc_open maps another
 * process's handle into this one on `device` (*dptr out = the allocation's
 * base: add the exporter's offset; close with cc_ipc_close).  Errors:
 * INVALID_ARG, UNSUPPORTED (no P2P path), CUDA. */
cc_status cc_peer_access(int32_t device, int32_t peer);

/* L2 residency for the reused operand (S§8(f)2; SpMV's x): set an
 * access-policy window on `stream` so later launches on it (also when
 * captured into a graph) mark [ptr, ptr + bytes) persisting in L2 with
 * `hit_ratio` in (0, 1], after raising the device's persisting-L2 limit to
 * cover it (clamped to the device maximum).  bytes = 0 clears the window and
 * resets the persisting lines.  Errors: INVALID_ARG, CUDA. */
cc_status cc_l2_persist(void* stream, const void* ptr, size_t bytes, float hit_ratio);
cc_status cc_ipc_handle(const void* dptr, void* handle64, uint64_t* offset);
cc_status cc_ipc_open(const void* handle64, int32_t device, void** dptr);
cc_status cc_ipc_close(void* dptr);

/* 2D cross-correlation (R15) with a (2R+1)^2 filter w (HOST, copied into the
 * launch parameters), R in {1, 3}; out = 0 outside [R, rows-R) x [R, cols-R).
 * in/out rows x cols fp32 DEVICE, leading dim ld (% 4 == 0).  Logical CTA = 32x32
 * output tile; grid ceil(cols/32) x ceil(rows/32). */
typedef struct { const float* in; float* out; int64_t ld; int32_t rows, cols; int32_t R; const float* w; } cc_conv2d_args;
/* CSR SpMV y = A x (R16).  DEVICE row_ptr[rows+1], col[nnz], val[nnz], x[cols],
 * y[rows] (zeroed by the call), int32 indices, nnz < 2^31.  Logical CTA b owns
 * the merge-path diagonals [4096 b, 4096 (b+1)) of the row-ends x nonzeros merge
 * grid (so power-law rows are balanced); grid = ceil((rows+nnz)/4096) x 1.
 * part (DEVICE, grid+1 entries) is the split table cc_spmv_partition fills once
 * per matrix structure.
 * Hub-column form (n_hot > 0, the output of cc_spmv_inspect): `col` holds the
 * inspector's encoding -- a reference to hub slot k is stored as -(k+1), any
 * other column as itself -- `hot` (DEVICE int32[n_hot]) the column of each
 * slot and `xh` (DEVICE float[n_hot], caller-owned scratch) receives the hub
 * values: each launch first gathers xh[n_hot-1-k] = x[hot[k]] (one small
 * kernel, counted in *launches), then the SpMV reads hub references from that
 * dense 4 * n_hot-byte array, which every SM keeps in L1.  Same y bits as the
 * plain form (the products and their order do not change).  n_hot = 0: plain
 * CSR, hot/xh ignored.
 * CC_K_SPMV_SHUB: the same computation and y bits, for the persistent
 * backends only (agent / identity / static; others UNSUPPORTED): each agent
 * copies the CC_SPMV_SHUB_SLOTS hottest hub values (slots 0 .. , the
 * inspector numbers slots in non-increasing degree order) into its shared
 * memory once, with one bulk copy when its first task is staged, and every
 * logical CTA it runs reads them from there (LDS) instead of through L1 / L2;
 * slots past the tier are read from xh as in the plain hub form.  The hub
 * columns are the x entries all logical CTAs share (inter-CTA reuse
 * of the data-related class), caught on chip by the persistent agent.
 * xh 16-byte aligned. */
#define CC_SPMV_SHUB_SLOTS 8192
typedef struct { int32_t rows, cols; int64_t nnz; const int32_t* row_ptr; const int32_t* col;
                 const float* val; const float* x; float* y; const int32_t* part;
                 const int32_t* hot; float* xh; int32_t n_hot; } cc_spmv_args;
/* CC_K_HIST64 -- 64-bin histogram, the paper's HST (Table 2; data-
 * related); reading R24 (CUDA SDK histogram64):
 *     counts[k] = #{ i < n : data[i] >> 2 == k },  k = 0..63.
 * data: DEVICE, n bytes, 16-byte aligned; counts: DEVICE uint32[64], zeroed by
 * the call (cudaMemsetAsync on `stream`) then accumulated; 0 <= n < 2^32.
 * Logical CTA b counts the 32 KiB chunk [32768 b, 32768 (b+1)); grid =
 * ceil(n / 32768) x 1.  Persistent agents keep per-warp shared sub-histograms
 * across their chunks and flush once; one-shot CTAs flush per chunk. */
typedef struct { const uint8_t* data; int64_t n; uint32_t* counts; } cc_hist64_args;

/* Fill args->part-sized DEVICE table `part` (gx+1 entries, gx from
 * cc_kernel_grid) with the merge-path row coordinate of each logical CTA's
 * first diagonal.  Asynchronous on `stream`. */
cc_status cc_spmv_partition(const cc_spmv_args* args, int32_t* part, void* stream);

/* Inspector for the data-related class ("a lightweight inspector
 * kernel before runtime to profile local data access ... in order to predict
 * global data organization"): find the (up to) max_hot most-referenced
 * columns of the plain CSR in `args` (args->col, args->cols; n_hot ignored)
 * and write the hub-column form: hot[slot] = column (DEVICE int32[max_hot]),
 * col_hot[k] = -(slot+1) for a hub reference, else col[k] (DEVICE int32[nnz];
 * may not alias col).  scratch: DEVICE int32[cols + 65536 + 2].  Columns with
 * no reference are never hubs; ties at the degree threshold are taken in an
 * unspecified order.  Slots [0, min(n_hot, CC_SPMV_SHUB_SLOTS)) hold the most
 * referenced hubs (every one referenced at least as often as any later slot;
 * degrees clamped at 65535), the rest the others; inside each range slots
 * follow column order only roughly (they are handed out by atomic counters),
 * which keeps a row's sorted column run on few lines of the hub array.
 * *n_hot (HOST) = slots used.  Runs on `stream` and
 * synchronizes it (one 256 KB degree histogram is read back to pick the
 * threshold).  Errors: INVALID_ARG (null, max_hot < 0), CUDA. */
cc_status cc_spmv_inspect(const cc_spmv_args* args, int32_t max_hot, int32_t* hot, int32_t* col_hot,
                          int32_t* scratch, int32_t* n_hot, void* stream);

/* Listing 3 microbenchmark (section 3.1): `ctas` one-warp CTAs
 * in hardware order; thread 0 of CTA b times one L1-allocating load
 * (plain ld.global -> LDG.E) of input[32 * smid] -- the address depends only on the SM,
 * so only CTAs on the same SM can share the line -- optionally after spinning
 * `stagger_cycles * b` cycles (the STAGGERED variant, l.7-9).  All pointers
 * DEVICE, caller-owned: input >= 32 * smid_span floats (cc_device_info);
 * outputs smid[ctas] (%smid of CTA b), ticks[ctas] (%clock64 cycles of the
 * load), sink[ctas] (loaded value + 1; keeps the load alive).  Asynchronous on
 * `stream`.  ctas < 0, stagger_cycles < 0 or a NULL pointer with ctas > 0:
 * CC_ERR_INVALID_ARG; ctas == 0 is a no-op. */
cc_status cc_l1_reuse_probe(int32_t ctas, int32_t stagger_cycles, const float* input, int32_t* smid,
                            uint32_t* ticks, float* sink, void* stream);

/* Logical grid a kernel needs for `args` (so the caller can build the plan). */
cc_status cc_kernel_grid(int32_t kernel, const void* args, int32_t* gx, int32_t* gy);
/* Occupancy limit (agents per SM) of `kernel`'s agent body on `device`
 * (CC_K_JACOBI5_WAVE: worker warps per SM at fuse = 4; 24 / 20 / 15 for
 * fuse <= 3 / 4 / 5-8). */
cc_status cc_max_agents(int32_t kernel, int32_t device, int32_t* max_agents);

/* Run `kernel` over the plan's logical grid with the chosen backend, on
 * `stream`.  The plan's grid must equal cc_kernel_grid(kernel, args).  The
 * agent backends use the plan's workspace, which resets itself at the end of
 * each launch, so launches sharing a plan never overlap: an agent or identity
 * launch on a stream other than the previous launch's is made to wait for
 * that launch's completion (cudaStreamWaitEvent, recorded under the plan's
 * mutex together with the launch, so concurrent host threads are safe too).
 * Use a second plan for concurrency.  Launches being captured into a CUDA
 * graph are neither ordered nor recorded: the capturing code orders them.
 * The calling thread's current device is unchanged on return (also on errors).
 * `launches` (HOST, optional) receives the number of kernels this call queued. */
cc_status cc_launch(cc_plan plan, int32_t kernel, const void* args,
                    const cc_launch_opts* opts, void* stream, int32_t* launches);

/* ---------------------------------------------------------------------------
 * Multi-GPU exchange steps (S§8(e)): one process per GPU, NCCL over NVLink /
 * NVSwitch.  NCCL is resolved at run time (the copy the process already maps,
 * e.g. PyTorch's, or the file named by CC_NCCL_LIBRARY); without it these
 * return CC_ERR_UNSUPPORTED.  All are asynchronous on `stream`.
 * ------------------------------------------------------------------------- */
typedef struct cc_comm_s* cc_comm;
/* Rank 0 creates the 128-byte NCCL unique id (HOST out) and shares it with the
 * other ranks out of band (e.g. a torch.distributed broadcast). */
cc_status cc_comm_unique_id(void* id128);
/* Collective over all ranks: communicator of `nranks`, this process is `rank`
 * on CUDA `device`.  Errors: INVALID_ARG, UNSUPPORTED (no NCCL), NCCL. */
cc_status cc_comm_init(const void* id128, int32_t nranks, int32_t rank, int32_t device, cc_comm* comm);
cc_status cc_comm_destroy(cc_comm comm);
/* Slab halo exchange for the sharded stencils: `slab` (DEVICE, rows x cols fp32,
 * leading dim ld) holds this rank's owned rows plus `halo` rows above (unless
 * rank 0) and below (unless the last rank); the halo rows are overwritten with
 * the neighbours' owned boundary rows (one grouped send/recv per neighbour). */
cc_status cc_halo_exchange(cc_comm comm, float* slab, int64_t ld, int32_t rows, int32_t cols, int32_t halo,
                           void* stream);
/* In-place sum over ranks of `count` fp32 (DEVICE): the transposed products of
 * the row-sharded ATAX family. */
cc_status cc_allreduce_sum(cc_comm comm, float* buf, size_t count, void* stream);
/* Gather `count_per_rank` fp32 from every rank, rank-major into recv (DEVICE). */
cc_status cc_allgather(cc_comm comm, const float* send, float* recv, size_t count_per_rank, void* stream);

/* Messages. */
const char* cc_status_string(cc_status s);
const char* cc_last_error(void);       /* thread-local detail of the last failure */
int         cc_last_cuda_error(void);  /* cudaError_t behind the last CC_ERR_CUDA */
const char* cc_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CTACLUST_H */
