/*
 * graffix.h -- C ABI of libgraffix.so, the B200-native hot path of Graffix
 * (Singh & Nasre, "Graffix: Efficient Graph Processing with a Tinge of
 * GPU-Specific Approximations", ICPP 2020).  Citations "P@N" refer to
 * /root/reference/PAPER.md (one physical line), character offset N.
 *
 * The path: upload a CSR graph (P@15127, §2.1 Fig 1),
 * transform it with the three Graffix techniques (Alg 2 P@16373 coalescing;
 * §3 P@29857 shared memory; §4 P@33145 divergence), then run the iterative
 * vertex-centric sweeps ("main fixed-point loop repeatedly calling the
 * primary kernel", P@40883) for SSSP / PageRank / SCC / MST / BC
 * (P@36969), merging replica copies after every iteration (§2.4 P@28309),
 * and download per-vertex results in ORIGINAL vertex ids.
 *
 * Conventions
 *  - Plain C: no C++ or torch types cross this boundary.  Every function
 *    returns gx_status (or a plain value) and never throws; on failure
 *    gx_last_error() returns a thread-local message valid until the next
 *    gx_* call on the same thread, and the object is left in its previous
 *    valid state.
 *  - Ownership: the library copies every input; callers keep their arrays.
 *    All device memory is owned by the library (allocated through the hook
 *    of gx_set_allocator, else cudaMallocAsync on the context's stream) and
 *    released by the matching destroy call.
 *  - Threads: one gx_graph is used by one host thread at a time.
 *  - Multi-GPU: one gx_ctx per rank (gx_ctx_create_dist); every rank calls
 *    every gx_* function collectively, in the same order, with the same
 *    arguments.
 *  - No CPU fallback: without a CUDA device the compute calls return
 *    GX_E_CUDA.
 */
#ifndef GRAFFIX_H
#define GRAFFIX_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GX_ABI_VERSION 1

typedef enum {
  GX_OK = 0,
  GX_E_INVALID = 1,     /* bad argument (range, monotonicity, knob bounds)     */
  GX_E_STATE = 2,       /* call out of order (run before upload, ...)          */
  GX_E_OOM = 3,         /* device or host allocation failed                    */
  GX_E_CUDA = 4,        /* CUDA runtime error or no device                     */
  GX_E_NCCL = 5,        /* NCCL error or library not loadable                  */
  GX_E_UNSUPPORTED = 6  /* e.g. (n-1)*max(w) >= 2^32-1, m' >= 2^32            */
} gx_status;

typedef enum { GX_SSSP = 1, GX_PAGERANK = 2, GX_SCC = 3, GX_MST = 4, GX_BC = 5 } gx_algo;

/* Confluence operator (§2.4, P@28421-28736): the paper's algorithm-agnostic
 * arithmetic mean, or the algorithm-aware one (SSSP: min of the copies;
 * PageRank: the owner's new value broadcast to its replicas). */
typedef enum { GX_MERGE_MEAN = 0, GX_MERGE_MIN = 1 } gx_merge;

/* Sweep mapping.  LB: edge-balanced warp-cooperative kernels (the best exact
 * kernels).  TPV: the paper's vertex-centric mapping, one thread per slot
 * (P@15381), lanes of a warp = 32 consecutive entries of the §4 schedule,
 * edges in SELL-32 slabs.  PB (PageRank only; other algorithms run LB):
 * propagation-blocked pull -- the x_u/D_u terms of the sum in P@36969 are
 * streamed along the edges in (source block, sink block) segments and summed
 * in shared memory, so no random global gathers remain; single GPU,
 * asynchronous schedule.  AUTO = the mapping measured fastest on B200 for
 * every configuration (exact and every knob): PB for PageRank
 * on one GPU when the graph spans at least GX_PB_MIN_BINS_PER_SM blocks of
 * 16384 slots per SM (with or without §3 tiles), else LB; LB for every other
 * algorithm.  TPV stays available as the paper's own mapping. */
/* VNS (the paper's second workload P@11477-11746: Graffix
 * layouts under another engine's mapping): Tigr-style virtual node splitting
 * on our own kernels -- every slot's out-row is cut into virtual nodes of at
 * most K edges (env GX_VNS_K, default 8), one thread per virtual node in the
 * TPV lane order (§4 schedule or slot order), so a warp's longest row is
 * bounded by K.  SSSP; PageRank runs TPV under it (a pull row cannot be split
 * without a combine step). */
typedef enum { GX_MAP_AUTO = 0, GX_MAP_LB = 1, GX_MAP_TPV = 2, GX_MAP_PB = 3, GX_MAP_VNS = 4 } gx_mapping;
#define GX_PB_MIN_BINS_PER_SM 1

/* upload / download flags */
#define GX_PTRS_HOST 0u       /* pointers are host memory (pageable or pinned)   */
#define GX_PTRS_DEVICE 1u     /* pointers are device memory of the ctx device    */
#define GX_VALIDATE 2u        /* check monotone row_ptr, col range, weights >= 1 */
#define GX_CANONICAL 4u       /* caller asserts: no self-loops, no duplicates    */
#define GX_DL_ASYNC 16u       /* gx_download: see there                          */
#define GX_W_U8 32u           /* gx_graph_upload_csr: w points to uint8_t weights
                                 (1..255), widened to 32 bits on the device: a
                                 quarter of the weights' PCIe bytes; device
                                 pointers need GX_CANONICAL                      */
#define GX_ASYNC_UPLOAD 8u    /* with GX_CANONICAL and host pointers, no GX_VALIDATE:
                                 the weights are copied on a second stream; see below */

/* download kinds */
#define GX_OUT_DIST_U32 1        /* SSSP distance, 0xFFFFFFFF = unreachable [n]  */
#define GX_OUT_RANK_F64 2        /* PageRank [n]                                  */
#define GX_OUT_LABEL_I32 3       /* SCC label = min original id in the SCC [n]    */
#define GX_OUT_BC_F64 4          /* betweenness (sampled sources) [n]             */
#define GX_OUT_MST_WEIGHT_U64 5  /* minimum spanning forest weight [1]            */

typedef struct gx_ctx gx_ctx;
typedef struct gx_graph gx_graph;

/* Knobs.  Every threshold is converted once to integer parts-per-million
 * (floor(x*1e6 + 0.5)) so that the host transforms compare exactly. */
typedef struct {
  uint32_t struct_size;          /* = sizeof(gx_knobs)                                */
  int32_t coalesce;              /* §2 on/off (Alg 2, P@16373)                        */
  int32_t chunk_k;               /* k in 1..32, default 16 (P@25752)                  */
  double replicate_threshold;    /* connectedness >= theta (P@24839); default 0.6;
                                    > 1 => renumber only                              */
  int32_t merge_op;              /* gx_merge, default GX_MERGE_MEAN                   */
  int32_t smem;                  /* §3 on/off (P@29857)                               */
  double cc_threshold;           /* CC > theta_cc (strict), default 0.5               */
  int64_t added_edge_budget;     /* §3 global limit, directed edges; < 0 => m/100     */
  int32_t smem_iters;            /* t; 0 => 2 * diameter of the subgraph (P@32282)    */
  int32_t smem_max_nodes;        /* S_max, default 64 (<= 255)                        */
  int32_t degree_norm;           /* §4 on/off (P@33145)                               */
  double degsim_threshold;       /* degreeSim < theta_d (strict), default 0.3         */
  double degree_target;          /* "degree-normalisation factor", default 0.85       */
  int32_t added_weight_rule;     /* weight of every added edge standing for a 2-hop
                                    path with hop weights w1, w2:
                                    GX_W_SUM (default) w1 + w2 (P@34493, reading R17:
                                    never shorter than the path, SSSP stays exact);
                                    GX_W_MAX max(w1, w2), GX_W_MEAN max(1, (w1+w2)/2)
                                    ("one can choose an alternative", P@34692)        */
  int32_t sibling_undirected;    /* §3: 0 (default) sibling edges only along directed
                                    2-paths a->c->b (R23); 1 any two neighbours of c
                                    in the undirected CC view (P@29950), both
                                    directions, hop weights = lighter direction       */
} gx_knobs;

#define GX_W_SUM 0
#define GX_W_MAX 1
#define GX_W_MEAN 2

typedef struct {
  int64_t n_slots, n_holes, n_replicas, holes_filled;
  int64_t edges_added_coalesce, edges_added_smem, edges_added_degnorm;
  int64_t n_subgraphs, subgraph_vertices, m_slots;
  double transform_ms, extra_space_pct;
} gx_transform_info;

typedef struct {
  int32_t iterations;
  int32_t converged;       /* 1 fixed point reached (SSSP: empty frontier; PR: delta < tol),
                              0 max_iters hit, 2 PR stopped at the fp32-contrib noise floor */
  double loop_ms;          /* device time of init + fixed-point loop (CUDA events) */
  double last_delta;       /* PR: final L1 delta                                   */
  int64_t edges_scanned;   /* edges relaxed / gathered over all iterations         */
  int64_t bytes_model;     /* algorithmic bytes          */
  int64_t vertices_active; /* sum over iterations of active slots                  */
  int32_t kernel_launches; /* library kernels launched by this run                 */
  int32_t sweep_launches;  /* profile: launches of the main sweep kernel            */
  double sweep_ms;         /* profile: summed CUDA-event time of the main sweep kernel */
  int64_t sweep_bytes;     /* algorithmic bytes moved by the main sweep kernel       */
  int32_t mapping_used;    /* gx_mapping the sweeps ran with (AUTO resolved)         */
  int32_t dense_iterations; /* SSSP: iterations run as the blocked dense relaxation   */
} gx_run_info;

typedef struct {
  uint32_t struct_size;    /* = sizeof(gx_run_opts)                                */
  int32_t algo;            /* gx_algo                                              */
  int64_t source;          /* SSSP source (original id); < 0 => max out-degree (R36) */
  int32_t max_iters;       /* cap on fixed-point iterations (0 => 1000000)         */
  int32_t mapping;         /* gx_mapping                                           */
  double tol;              /* PR: stop when L1 delta < tol (default 1e-9)          */
  double damping;          /* PR: d (default 0.85)                                 */
  int32_t check_every;     /* host reads the convergence flag every c iterations   */
  int32_t use_graphs;      /* capture the c-iteration batch in a CUDA graph         */
  const int64_t* bc_sources; /* BC: host array of original ids                     */
  int64_t n_bc_sources;
  int32_t profile;         /* 1 => eager launches with a CUDA event pair around every
                              main sweep kernel (sweep_ms / sweep_launches below)   */
  int32_t sim_ranks;       /* > 1 on a single-GPU context: run the 1-D partitioned
                              path with this many simulated ranks (exchange by a
                              device reduction instead of NCCL); LB mapping only    */
  int32_t pr_schedule;     /* PR update schedule on one GPU (SURVEY §8(c) Theorem E3:
                              every schedule has the same fixed point x*):
                              GX_PR_ASYNC (default) = one contrib buffer updated in
                              place, a row reads whichever of x_t / x_{t+1} its
                              sources hold (asynchronous vertex-centric kernels,
                              P@15381), half the contrib footprint;
                              GX_PR_JACOBI = sweep t reads only x_t (two contrib
                              buffers, the oracle's iteration order).
                              Both scale iteration t's inputs by 1/sum(x_t) (lazy
                              normalisation; the fixed point sums to 1), without
                              which the asynchronous schedule and the §3 local
                              pass lose mass that decays only at rate d per
                              iteration (RMAT-24: async 14 iterations, Jacobi 22;
                              DESIGN.md R56).  The multi-GPU path is Jacobi.     */
  int32_t merge_every;     /* §2.4 confluence cadence (P@28188-28736):
                              1 (default) = after every iteration; c > 1 = after
                              every c-th iteration and once more whenever the
                              sweep alone has reached its fixed point; 0 = only
                              then ("merge at the end").  Every cadence ends at a
                              merged fixed point (Theorems E1/E3).                */
} gx_run_opts;

#define GX_PR_JACOBI 0
#define GX_PR_ASYNC 1

/* Transformed-graph export (debug / parity path).  Two-call protocol: call
 * gx_export_sizes, allocate host arrays of those sizes, call
 * gx_export_transformed; any pointer may be NULL to skip that array.  The
 * slot CSR rows are sorted by destination slot (reading R11). */
typedef struct {
  int64_t n_slots, m_slots, n_tiles, tile_members_len, sched_len;
} gx_export_sizes_t;

typedef struct {
  int64_t* row_ptr;        /* [n_slots+1]                                         */
  int32_t* col;            /* [m_slots] destination slot                          */
  uint32_t* w;             /* [m_slots]                                           */
  uint8_t* edge_added;     /* [m_slots] 0 original, 1 §2 2-hop, 2 §3, 3 §4        */
  int32_t* slot_to_orig;   /* [n_slots] -1 for holes                              */
  uint8_t* slot_kind;      /* [n_slots] 0 owner, 1 replica, 2 hole                */
  int32_t* sched;          /* [sched_len] lane -> slot (§4), identity otherwise   */
  int64_t* tile_ptr;       /* [n_tiles+1] into tile_members                       */
  int32_t* tile_members;   /* [tile_members_len] original ids, ascending per tile */
  int32_t* tile_centre;    /* [n_tiles]                                           */
  int32_t* tile_iters;     /* [n_tiles] t                                         */
} gx_export_t;

int gx_abi_version(void);
const char* gx_last_error(void);

/* Context on CUDA device `device`; cuda_stream NULL => the library creates
 * its own non-blocking stream; otherwise all work is ordered on it. */
gx_status gx_ctx_create(gx_ctx** out, int device, void* cuda_stream);

/* Multi-GPU: rank 0 calls gx_get_nccl_unique_id and broadcasts the 128 bytes
 * (the binding uses torch.distributed); every rank then calls
 * gx_ctx_create_dist.  NCCL is dlopen'ed (torch's bundled libnccl.so.2). */
gx_status gx_get_nccl_unique_id(uint8_t out[128]);
gx_status gx_ctx_create_dist(gx_ctx** out, int device, void* cuda_stream, int rank,
                             int world, const uint8_t id[128]);

/* Hosted exchange: the same 1-D partitioned path (the paper
 * itself is single-GPU, P@38588) with a transport supplied by the caller
 * instead of NCCL -- e.g. torch.distributed over gloo, so that two processes
 * sharing ONE GPU run the library's real partitioned code.  Every collective
 * of the partitioned path is staged through a pinned host buffer owned by the
 * context: the library copies the device data to host_buf, calls fn, and
 * copies the part it relies on back.  fn must return 0 on success (any other
 * value fails the run with GX_E_NCCL) and must be called collectively by
 * every rank (same kind / count / dtype / op / offsets):
 *   GX_COLL_ALLREDUCE       host_buf[0..count) <- reduction (op) over ranks
 *   GX_COLL_ALLGATHERV      host_buf[offsets[r]..offsets[r+1]) <- rank r's
 *                           values of that slice, for every r (count =
 *                           offsets[world]; offsets has world+1 entries)
 *   GX_COLL_REDUCE_SCATTERV host_buf[offsets[rank]..offsets[rank+1]) <- the
 *                           reduction over ranks of that slice (only this
 *                           slice is read back)
 * dtype: GX_DT_U32 / GX_DT_F32 / GX_DT_F64; op: GX_OP_SUM / GX_OP_MIN.
 * Errors: GX_E_INVALID (fn NULL, rank outside [0, world)), GX_E_CUDA. */
#define GX_COLL_ALLREDUCE 0
#define GX_COLL_ALLGATHERV 1
#define GX_COLL_REDUCE_SCATTERV 2
#define GX_DT_U32 0
#define GX_DT_F32 1
#define GX_DT_F64 2
#define GX_OP_SUM 0
#define GX_OP_MIN 1
typedef int (*gx_coll_fn)(int32_t kind, void* host_buf, int64_t count, int32_t dtype, int32_t op,
                          const int64_t* offsets, int32_t world, void* user);
gx_status gx_ctx_create_hosted(gx_ctx** out, int device, void* cuda_stream, int rank, int world,
                               gx_coll_fn fn, void* user);

/* Device allocator hook (e.g. torch's caching allocator).  alloc returns a
 * device pointer or NULL; release frees it.  Must be set before uploads. */
typedef void* (*gx_alloc_fn)(size_t bytes, void* stream, void* user);
typedef void (*gx_release_fn)(void* ptr, size_t bytes, void* stream, void* user);
gx_status gx_set_allocator(gx_ctx* ctx, gx_alloc_fn alloc, gx_release_fn release, void* user);
void gx_ctx_destroy(gx_ctx* ctx);
gx_status gx_ctx_stream(gx_ctx* ctx, void** stream_out);

/* Upload a directed CSR graph (P@15127): row u = col[row_ptr[u]..row_ptr[u+1]),
 * weights w (NULL => all 1; must be >= 1).  Canonicalised (reading R2): self-
 * loops dropped, a duplicate (u,v) merged into its first occurrence keeping
 * the minimum weight, row order otherwise kept -- unless GX_CANONICAL.
 * GX_ASYNC_UPLOAD (with GX_CANONICAL, host pointers, w != NULL, no GX_VALIDATE;
 * ignored otherwise): the call returns once row_ptr and col are queued; w is
 * copied on a second stream behind col, so a following exact-mode PageRank on
 * the blocked mapping (which needs only the structure) overlaps its transfer.
 * The caller keeps row_ptr / col / w valid and unchanged until a call that
 * joins the copy: gx_run of any other algorithm or mapping, gx_transform,
 * gx_export_*, gx_sync or gx_graph_destroy.  Pinned host memory is needed for
 * the copies to overlap anything.
 * GX_W_U8: w is read as m uint8_t values (the paper-style weights 1..100 fit).
 * Errors: GX_E_INVALID (n < 0, m < 0, with GX_VALIDATE: non-monotone row_ptr,
 * col out of [0,n), w = 0), GX_E_UNSUPPORTED (m >= 2^32 or n >= 2^31). */
gx_status gx_graph_upload_csr(gx_ctx* ctx, gx_graph** out, int64_t n, int64_t m,
                              const int64_t* row_ptr, const int32_t* col, const uint32_t* w,
                              uint32_t flags);
void gx_graph_destroy(gx_graph* g);

/* Host-only graph: canonicalised as above, no device memory.  gx_transform
 * and the gx_export_* calls work on it (the transforms are host code);
 * gx_run / gx_download return GX_E_STATE.  Used by the CPU test suite. */
gx_status gx_graph_create_host(gx_graph** out, int64_t n, int64_t m, const int64_t* row_ptr,
                               const int32_t* col, const uint32_t* w, uint32_t flags);
gx_status gx_graph_info(gx_graph* g, int64_t* n, int64_t* m);

/* Paper defaults, all techniques OFF (= exact mode). */
gx_status gx_knobs_default(gx_knobs* k);

/* The transforms §2 -> §3 -> §4 (composition reading R34) and the device
 * layouts they need; with a device context the slot graph is built in HBM
 * (SURVEY §8(f) N1), only the sequential steps run on the host.  NULL knobs => exact mode (identity).
 * With env GX_TRANSFORM_FREE_LAYOUTS=1 the graph's previous device layouts
 * and results are released before the transform runs (their memory is needed
 * for the edge lists at RMAT-26 scale).
 * Errors: GX_E_INVALID (k not in 1..32, thresholds not in [0,1] except
 * replicate_threshold >= 0, degree_target not in (0,1], smem_max_nodes not
 * in 2..255); GX_E_OOM / GX_E_CUDA from the device pipeline, after which the
 * graph is back in exact mode. */
gx_status gx_transform(gx_graph* g, const gx_knobs* knobs, gx_transform_info* info);

gx_status gx_export_sizes(gx_graph* g, gx_export_sizes_t* sizes);
gx_status gx_export_transformed(gx_graph* g, gx_export_t* out);

/* Run one algorithm to its fixed point on the transformed graph.  Not
 * converging within max_iters is not an error (converged = 0).  On a
 * partitioned context (world > 1): SSSP and PageRank sweep the
 * rank's rows and exchange after every sweep; BC is source-parallel (rank p
 * takes sources p, p+P, ..., then one allreduce(sum) of bc); SCC and MST sweep
 * the rank's share of the logical edges and reduce the per-vertex colours /
 * per-component proposals over the ranks every round.  Every rank returns the
 * whole result.
 * Errors: GX_E_STATE (no graph), GX_E_INVALID (source out of range),
 * GX_E_UNSUPPORTED (SSSP: a shortest-path length reached 2^32-2, the saturation
 * value of the uint32 distances, reading R51; the result is then not valid). */
gx_status gx_run(gx_graph* g, gx_algo algo, int64_t source, int32_t max_iters, double tol,
                 gx_run_info* info);
gx_status gx_run_ex(gx_graph* g, const gx_run_opts* opts, gx_run_info* info);
gx_status gx_run_opts_default(gx_run_opts* o);

/* Copy a result (indexed by ORIGINAL vertex id; owner slots after the final
 * merge) into `out` (host or device per flags).  count = n, or 1 for MST.
 * GX_DL_ASYNC (distances / ranks of an untransformed graph into host memory;
 * ignored otherwise): the copy is queued on a second stream behind the run
 * that produced the result and the call returns at once, so a following run
 * of another algorithm overlaps it.  `out` is complete after gx_sync, and is
 * also waited for by the next run that overwrites that result, by gx_transform
 * and by gx_graph_destroy; do not read it before.  Pinned memory for overlap.
 * Errors: GX_E_STATE (that algorithm has not run), GX_E_INVALID (count). */
gx_status gx_download(gx_graph* g, int32_t kind, void* out, int64_t count, uint32_t flags);

/* 1-D partition used by the multi-GPU path: bounds[0..P]
 * over rows [0,n) of the host CSR row_ptr, balancing (edges + rows) per rank,
 * each interior bound rounded to a multiple of `align` (the PR window, 1024).
 * Host-only; no device needed.  Errors: GX_E_INVALID (P < 1, align < 1). */
gx_status gx_partition_rows(int64_t n, const int64_t* row_ptr, int32_t P, int64_t align, int64_t* bounds);

/* Synchronise the context stream (host wait). */
gx_status gx_sync(gx_ctx* ctx);

#ifdef __cplusplus
}
#endif
#endif /* GRAFFIX_H */
