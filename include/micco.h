/*
 * include/micco.h — C-ABI of the B200-native MICCO correlator engine.
 *
 * What it computes (PAPER.md, "MICCO", IPDPS'22):
 *   A many-body correlation function is "a sum of a large number of contraction
 *   terms each of which can be represented by a graph" (§Abstract).  Each
 *   graph's vertices are the quarks (legs) of hadron nodes, its edges quark
 *   propagations (L11, L17, L50); hadron nodes are batched matrices (mesons)
 *   or rank-3 tensors (baryons) over many time slices (L50, L54).  A graph is
 *   contracted by reducing "one edge after another", each reduction a tensor
 *   contraction between hadron nodes (L17-19, L56-60).  This library returns
 *       C(t) = Σ_g c_g · val_g(t),   t = 0 .. Lt-1,
 *   val_g(t) = Σ_{σ: edges → index} Π_instances T[t][σ(legs)].
 *   Repeated nodes and shared intermediates are computed once (L23, L71); the
 *   pairwise contractions are scheduled over GPUs with the paper's reuse-aware
 *   heuristic (Alg. 1/2, L203-288) under reuse bounds (L150, Table II).
 *
 * Element type: complex double.  At this boundary tensors are interleaved
 * (re, im) doubles, row-major over [Lt][N]...[N] (t slowest), i.e.
 * 2 * Lt * N^rank doubles per node (SURVEY.md §8(c) readings #2, #3).
 *
 * Conventions for every call:
 *  - Returns micco_status (0 = OK).  Nothing throws or aborts across the ABI.
 *  - micco_last_error(ctx) describes the last failure on that ctx.
 *  - The caller owns every pointer it passes; the library copies what it keeps
 *    before returning.  The library owns all pinned host and device memory it
 *    allocates; micco_destroy releases it.
 *  - A context is not thread-safe; distinct contexts are independent.
 *  - CUDA/NCCL failures return MICCO_ERR_CUDA / MICCO_ERR_NCCL and make the
 *    context unusable ("sticky"), except for micco_destroy / micco_last_error.
 *  - Creating a context and adding nodes/graphs needs no GPU; micco_execute
 *    needs one (there is no CPU fallback: without a CUDA device it returns
 *    MICCO_ERR_CUDA).
 */
#ifndef MICCO_H
#define MICCO_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define MICCO_API __attribute__((visibility("default")))
#else
#define MICCO_API
#endif

typedef struct micco_ctx micco_ctx;

typedef enum {
  MICCO_OK = 0,
  MICCO_ERR_ARG = -1,          /* null pointer, bad size, Lt mismatch, n_gpus out of range */
  MICCO_ERR_STATE = -2,        /* e.g. get_correlator before execute; sticky context */
  MICCO_ERR_GRAPH = -3,        /* invalid graph: leg unmatched / matched twice / index >= rank,
                                  joined legs with unequal N, order not a permutation */
  MICCO_ERR_UNSUPPORTED = -4,  /* intermediate rank > 4, baryon partial trace */
  MICCO_ERR_OOM = -5,          /* host or device memory, or a working set above the budget */
  MICCO_ERR_CUDA = -6,
  MICCO_ERR_NCCL = -7,
  MICCO_ERR_RANGE = -8         /* t outside [0, Lt) */
} micco_status;

/* leg p of instance u <-> leg q of instance v (one quark propagation) */
typedef struct {
  int32_t u, p, v, q;
} micco_edge;

/* Scheduling policies.  MICCO = Alg. 1 + Alg. 2 with the given reuse bounds
 * (PAPER.md L195-288); MICCO_NAIVE = bounds forced to (0,0,0) (L312);
 * ROUND_ROBIN = pair i of a vector to GPU i mod n; LEAST_LOADED = the GPU with
 * the least accumulated computation ("earliest available device", the Groute
 * rule of L312/L400); MICCO_AFFINITY = MICCO, except that when the GPU that last
 * consumed the pair's first operand (else its second) is in Alg. 1's candidate queue,
 * Alg. 2 takes it instead of the least-loaded candidate (not in the paper: once replicas
 * of a tensor exist on several GPUs, least-computation alternates its consumers between
 * them and spreads the replicas further; the candidate queue still bounds the imbalance). */
enum {
  MICCO_POLICY_MICCO = 0,
  MICCO_POLICY_MICCO_NAIVE = 1,
  MICCO_POLICY_ROUND_ROBIN = 2,
  MICCO_POLICY_LEAST_LOADED = 3,
  MICCO_POLICY_MICCO_AFFINITY = 4
};

typedef struct {
  size_t struct_size;          /* sizeof(micco_options): ABI versioning */
  int64_t mem_budget_bytes;    /* per GPU (GPUMaxMemory); 0 = device free memory
                                  minus a 2 GiB reserve, split evenly between logical GPUs
                                  sharing a device (multi-process mode: the minimum over ranks,
                                  agreed by an NCCL all-reduce, so every rank plans alike) */
  int32_t policy;              /* MICCO_POLICY_* */
  int32_t window_graphs;       /* graphs per window (one stream of vectors); 0 = auto: the largest
                                  of 256·n_gpus, 128·n_gpus, ..., 1 whose plan a smaller window does not beat by
                                  more than 1% in the planner's cost model, stopping at the first
                                  plan without D2H spills (a window's first-level intermediates
                                  are live together, so a tight budget needs a small window) */
  uint64_t seed;               /* tie-break RNG seed when deterministic == 0 */
  int32_t deterministic;       /* 1 (default) = lexicographic tie-breaks */
  int32_t keep_inputs_resident;/* 1 = node tensors uploaded by execute stay cached on the GPUs for
                                  the next execute (the "inputs resident in HBM" measurement);
                                  released by micco_release_cache or destroy */
  int32_t dist_rank;           /* multi-process mode: this process's rank (one process per GPU); */
  int32_t dist_world;          /*   world size, 0 = single-process mode (default) */
  int32_t reorder;             /* 1 = reuse-aware reduction order for every graph added from now on
                                  (SURVEY.md §8(f) NEXT #3): the caller's order is ignored and each
                                  step takes an already-interned contraction when one exists, else
                                  the smallest result, fewest flops, fewest hadron nodes (so
                                  node-pair products, the most shareable, come first), lowest
                                  edge.  0 (default) = the caller's order, greedy when NULL */
  int32_t bound_model;         /* how execute(reuse_bound = NULL) picks the reuse bounds on more than
                                  one GPU: 0 (default) one set for the whole plan, the cheapest of
                                  {0,1,2}^3 under the planner's cost model; 1 a set per vector
                                  (stage), the cheapest for that vector; 2 a set per vector from the
                                  fitted regression (a random forest over vector
                                  features, trained offline on mode-1 choices by
                                  tools/train_bounds.py) */
  int32_t scalar_tables;       /* where rank-0 results (per-slice scalars) are written before the
                                  final cross-GPU reduce: 0 (default) one table per CUDA device;
                                  1 one table per logical GPU, so the combine (peer copy + exact
                                  accumulate, every slot nonzero in one table only) runs even when
                                  several logical GPUs share a device.  C(t) is bitwise the same */
} micco_options;

/* Fill *opt with the defaults (struct_size set). */
MICCO_API void micco_options_default(micco_options *opt);

/* Create a context.  opt NULL = defaults.  No GPU is touched. */
MICCO_API micco_status micco_create(micco_ctx **out, const micco_options *opt);

/* Destroy a context and every host/device resource it owns.  NULL-safe. */
MICCO_API void micco_destroy(micco_ctx *ctx);

/* Add a hadron node (a batched matrix or tensor).
 * rank: 2 (meson) or 3 (baryon); N: leg dimension (1..65536); Lt: time slices (equal for
 * every node of a context, else MICCO_ERR_ARG); data: 2*Lt*N^rank doubles (interleaved,
 * row-major, t slowest), copied into library-owned pinned host memory.
 * Nodes with identical content are deduplicated (64-bit content hash + memcmp): *node_id is
 * then the existing id.  Repeated hadron nodes are the paper's reuse source (L23, L71). */
MICCO_API micco_status micco_add_hadron_node(micco_ctx *ctx, int32_t rank, int32_t N, int32_t Lt,
                                             const double *data, int64_t *node_id);

/* Harness extension (not part of the paper's interface): add `count` nodes whose data is
 * the counter-based generator micco_inputs/synth.h (seed, keys[i], mode, scale), generated
 * directly into pinned memory by a host thread pool.  Dedup is by generator descriptor.
 * node_ids: count entries out. */
MICCO_API micco_status micco_add_hadron_nodes_synth(micco_ctx *ctx, int32_t count, int32_t rank,
                                                    int32_t N, int32_t Lt, uint64_t seed,
                                                    const uint64_t *keys, int32_t mode, double scale,
                                                    int64_t *node_ids);

/* Add a contraction graph.
 * n_inst instances; node_ids[u] is instance u's node.  edges: n_edges leg pairs forming a
 * perfect matching of all instance legs (else MICCO_ERR_GRAPH).  A self-edge is allowed only
 * as the full trace of a meson instance.  order: a permutation of [0, n_edges) giving the
 * reduction order (the sequence the upstream Redstar emits, L56), or NULL = greedy (smallest
 * intermediate, then fewest flops, then lowest edge index).  Reducing an edge that joins two
 * components contracts every edge between them; an intermediate of rank
 * > 4 is MICCO_ERR_UNSUPPORTED.  coef: the graph's complex coefficient c_g.
 * Shared pairwise contractions are hash-consed: the same (operands, contracted legs) is one
 * task however many graphs use it.  *graph_id (may be NULL) = index of the graph. */
MICCO_API micco_status micco_add_graph(micco_ctx *ctx, int32_t n_inst, const int64_t *node_ids,
                                       int32_t n_edges, const micco_edge *edges,
                                       const int32_t *order, double coef_re, double coef_im,
                                       int64_t *graph_id);

/* Evaluate the correlator on n_gpus GPUs (single-process mode: logical GPU g runs on CUDA
 * device g % device_count, so n_gpus may exceed the device count for testing; multi-process
 * mode: n_gpus must equal dist_world and this process drives device dist_rank % count).
 * reuse_bound: the three reuse bounds of Table II (L138-152), each in [0, n_tasks], or NULL =
 * choose by sweeping {0,1,2}^3 through the planner's cost model (the paper's offline labels,
 * L292).  Repeatable; each call recomputes from node tensors (caches are cold unless
 * keep_inputs_resident).  The result is the same C(t) for any n_gpus, bounds and policy. */
MICCO_API micco_status micco_execute(micco_ctx *ctx, int32_t n_gpus, const int32_t *reuse_bound);

/* C(t) of the last execute: out[0] = Re, out[1] = Im.  MICCO_ERR_STATE before any execute,
 * MICCO_ERR_RANGE for t outside [0, Lt). */
MICCO_API micco_status micco_get_correlator(const micco_ctx *ctx, int32_t t, double out[2]);

/* val_g(t) of the last execute (before the coefficient), 2 doubles. */
MICCO_API micco_status micco_get_graph_value(const micco_ctx *ctx, int64_t graph_id, int32_t t,
                                             double out[2]);

/* Message for the last failure on ctx ("" if none).  Valid until the next call on ctx. */
MICCO_API const char *micco_last_error(const micco_ctx *ctx);

typedef struct {
  size_t struct_size;
  double wall_ms;              /* micco_execute wall time */
  double sched_ms;             /* planning + scheduling (host) */
  double kernel_ms;            /* device time inside contraction kernels (CUDA events; the union
                                  of the launches' intervals per device, summed over devices) */
  double copy_ms;              /* device time of the timed H2D copies (same union rule) */
  int64_t bytes_h2d, bytes_p2p, bytes_d2h;
  int64_t evictions;           /* replicas dropped or spilled to make room */
  int64_t cache_hits;          /* operand uses served by a resident replica */
  int64_t unique_tasks;        /* pairwise contractions after hash-consing */
  int64_t dedup_hits;          /* graph steps served by an existing task */
  int64_t n_gemm, n_dot;       /* tasks by kind (GEMM-shaped with rank>0 result / scalar) */
  int64_t n_stages;            /* vectors executed */
  int64_t kernel_launches;     /* CUDA kernels launched by the last execute */
  double flops;                /* algorithmic flops of the executed unique tasks (8 per complex MAC) */
  double flops_no_dedup;       /* the same counted per graph, without dedup */
  double max_over_mean_load;   /* max/mean flops per GPU */
  int32_t reuse_bound[3];      /* bounds used (after auto-selection) */
  int32_t n_gpus;
  double gemm_kernel_ms;       /* device time of the GEMM launches only (CUDA events on the
                                  launching stream; union of their intervals: a chunk's launches
                                  overlap on two streams) */
  double dot_kernel_ms;        /* device time of the dot/trace launches only */
  int64_t gemm_launches, dot_launches;
  double gemm_flops;           /* algorithmic flops of the GEMM-shaped tasks executed */
  double dot_bytes;            /* algorithmic bytes read by the dot/trace tasks executed */
  double enqueue_ms;           /* host time spent replaying the plan (issuing copies/kernels) */
  int32_t host_pinned;         /* 1 if every node tensor lives in page-locked host memory */
  int32_t gemm_3m;             /* 1 if the GEMMs used 3 real DMMA products per complex MAC (Gauss) */
  double gemm_dmma_flops;      /* flops actually executed on the DMMA pipe by the GEMMs
                                  (= gemm_flops, or 6/8 of it with the 3M scheme) */
  double dot_main_ms;          /* device time of the standalone dot launches (flat and transposed
                                  dots of two tensors; not traces, not fused-dot partial sums) */
  double dot_main_bytes;       /* algorithmic bytes those dots read: 16 B per element of both
                                  operands, all Lt slices (the HBM roofline numerator) */
  int64_t dot_main_launches;
  double plan_ms;              /* host time of make_plan for this execute (overlapped with the
                                  replay when planning streams; sched_ms = the same) */
  int64_t gemm_tma_launches;   /* GEMM launches on the TMA warp-specialized kernel (the rest ran on
                                  the cp.async kernels: ragged k, odd rows, 6-D views) */
  double model_s;              /* the plan's modelled time (planner cost model, core.h kModel*):
                                  Σ over stages of max over GPUs of flops + host bytes + peer bytes
                                  times (copies serialised with the kernels: pessimistic) */
  double model_overlap_s;      /* the same with each GPU's copies overlapping its kernels:
                                  Σ over stages of max over GPUs of max(flops, host, peer) time */
  int64_t peak_bytes;          /* the plan's largest resident set on one GPU (its memory demand) */
  int32_t window_graphs;       /* the window the plan used (options.window_graphs or the auto choice) */
  int64_t component_dedup_hits;/* graph components reused whole because an earlier graph held the same
                                  hadron nodes wired the same way up to relabeling (canonical
                                  sub-network hashing: tr(ABC) = tr(BCA) costs one contraction) */
  int64_t alloc_retries;       /* device allocations that had to drain the streams first (the copy
                                  and peer streams ran ahead of frees still queued on the compute
                                  stream) */
} micco_stats;

MICCO_API micco_status micco_get_stats(const micco_ctx *ctx, micco_stats *out);

/* Drop every cached replica (inputs kept by keep_inputs_resident). */
MICCO_API micco_status micco_release_cache(micco_ctx *ctx);

/* Switch the scheduling policy (MICCO_POLICY_*) of an existing context, for policy comparisons
 * on one loaded graph set (§V-B).  Drops cached replicas, so the next
 * execute starts cold; bounds chosen by an earlier sweep are re-chosen for the new policy.
 * Multi-process mode: every rank must make the same call. */
MICCO_API micco_status micco_set_policy(micco_ctx *ctx, int32_t policy);

/* ---- multi-process mode (one process per GPU; torch.distributed is the plumbing) ----
 * Rank 0 calls micco_nccl_unique_id, broadcasts the 128 bytes, then every rank calls
 * micco_set_nccl_id before its first execute.  Every rank must add the same nodes and graphs
 * in the same order; the plan is computed identically on every rank and each rank executes
 * the tasks assigned to its GPU, exchanging operands with ncclSend/ncclRecv over NVLink and
 * combining the per-graph scalars with one ncclAllReduce. */
MICCO_API micco_status micco_nccl_unique_id(uint8_t out[128]);
MICCO_API micco_status micco_set_nccl_id(micco_ctx *ctx, const uint8_t id[128]);

/* ---- device probe (measurement tooling, not the paper's interface) ----
 * The FP64 tensor-pipe ceiling of the current CUDA device: a register-only loop of
 * mma.sync m8n8k4 f64 (SASS DMMA.8x8x4), 16 warps per SM on every SM, 8 independent
 * accumulator chains per warp, for about `seconds` of device time (one short burst launch
 * first, then back-to-back launches).  *burst_tflops = the best single launch,
 * *sustained_tflops = the whole run (bench.py's roofline denominator for kernels timed
 * inside a long step; MEASURED_PEAKS.json has no FP64 figure).  512 flops per DMMA. */
MICCO_API micco_status micco_probe_fp64_peak(double seconds, double *burst_tflops,
                                             double *sustained_tflops);

/* ---- introspection for host-side tests (no GPU needed) ---- */

/* Run builder + planner + scheduler only, as execute would, and fill the stats fields that do
 * not need a device (unique_tasks, dedup_hits, n_gemm, n_dot, n_stages, bytes_*, evictions,
 * cache_hits, flops, max_over_mean_load, reuse_bound).  mem_budget_bytes must be set (no
 * device is queried).  assign (optional, unique_tasks entries) receives the GPU of each task
 * in task-id order. */
MICCO_API micco_status micco_plan(micco_ctx *ctx, int32_t n_gpus, const int32_t *reuse_bound,
                                  micco_stats *out, int32_t *assign);

/* The plan itself, for host-side invariant checks: like micco_plan, then copies up to max_ops
 * operations as 4 int32 each (kind, gpu, src, id) in replay order — kind 0 H2D (id = tensor),
 * 1 P2P (src → gpu), 2 SPILL (D2H), 3 FREE (gpu −1 = the host spill copy), 4 COMPUTE
 * (id = task), 5 FLUSH.  *n_ops receives the full count.  fused (optional, unique_tasks entries)
 * receives, per task, the dot task fused into its epilogue or −1. */
MICCO_API micco_status micco_plan_ops(micco_ctx *ctx, int32_t n_gpus, const int32_t *reuse_bound,
                                      int64_t max_ops, int32_t *ops, int64_t *n_ops, int32_t *fused);

/* Per-vector reuse bounds.  Plans like micco_plan with bound_mode 0
 * (reuse_bound, or the whole-plan sweep when NULL), 1 (per-vector sweep) or 2 (per-vector
 * regression); copies, for up to max_stages stages in order, the 6 vector features (balanceNum =
 * ceil(pairs/n_gpus), log2 mean operand bytes, repeated rate, resident rate, n_gpus, memory
 * pressure = max resident/budget; taken before the vector is scheduled) into features[6*s..]
 * and the bounds used into bounds[3*s..].  *n_stages receives the stage count, *predicted_s
 * the plan's modelled time (max over GPUs per stage of flops/42.9 TF/s + host bytes/55.5 GB/s +
 * peer bytes/770 GB/s, summed over stages; core.h kModel*).  Needs options.mem_budget_bytes; no GPU. */
MICCO_API micco_status micco_plan_stages(micco_ctx *ctx, int32_t n_gpus, int32_t bound_mode,
                                         const int32_t *reuse_bound, int64_t max_stages,
                                         double *features, int32_t *bounds, int64_t *n_stages,
                                         double *predicted_s);

/* The fitted reuse-bound regression on one 6-feature vector (layout as micco_plan_stages):
 * raw[3] receives the forest's mean output, bounds[3] the rounded values clamped to [0, 2]. */
MICCO_API void micco_predict_bounds(const double *features, double *raw, int32_t *bounds);

/* The task DAG: per tensor its size in bytes (all Lt slices; 0 for per-slice scalars) and its
 * producing task (−1 for hadron nodes); per task (kind 0 GEMM / 1 dot / 2 trace, operand a,
 * operand b or −1, output tensor).  Arrays sized by *n_tensors / *n_tasks (query with NULL). */
MICCO_API micco_status micco_dag(const micco_ctx *ctx, int64_t *n_tensors, int64_t *n_tasks,
                                 int64_t *tensor_bytes, int32_t *tensor_task, int32_t *task_info);

/* The scheduler alone (Alg. 1 + Alg. 2) over a stream of vectors of tensor
 * pairs, with no eviction: pairs[7*i .. 7*i+6] = (tensor1, tensor2, out, flops, bytes1,
 * bytes2, bytes_out); vec_off[v] .. vec_off[v+1] are the pairs of vector v; resident holds
 * n_resident (tensor, gpu) pairs present before the first vector.  out_gpu receives the GPU of
 * every pair.  Used to check the native scheduler decision-for-decision against oracle/sched.py. */
MICCO_API micco_status micco_debug_schedule(int32_t n_gpus, const int32_t reuse_bound[3],
                                            double gpu_max_memory, int32_t n_vectors,
                                            const int64_t *vec_off, const double *pairs,
                                            int32_t n_resident, const int64_t *resident,
                                            int32_t *out_gpu);

#ifdef __cplusplus
}
#endif
#endif /* MICCO_H */
