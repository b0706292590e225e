// core.h — internal data model of the MICCO engine (host side).
//
// Tensors: hadron nodes (inputs) and the intermediates produced by pairwise
// hadron contractions (L17-19, L60) share one id space.  A Task is one unique pairwise
// contraction after hash-consing (shared reduction paths, L23).  Graphs keep the scalar
// tensors of their connected components and their coefficient.
#pragma once

#include <condition_variable>
#include <cstdint>
#include <cstring>
#include <memory>
#include <mutex>
#include <string>
#include <map>
#include <unordered_map>
#include <vector>

#include "micco.h"

namespace micco {

constexpr int kMaxRank = 4;  // intermediate rank cap

struct Error {
  micco_status code;
  std::string msg;
};

[[noreturn]] void fail(micco_status code, const std::string &msg);

struct NodeRec {
  int32_t rank = 0, N = 0;
  int64_t slice_elems = 0;  // N^rank complex elements per time slice
  double *host = nullptr;   // 2 * Lt * slice_elems doubles, interleaved, t slowest
  uint64_t hash = 0;
  int32_t tensor = -1;
  // generator descriptor of a synthetic node; in multi-process mode its data is generated on
  // first use by this rank (host == nullptr until then), so a rank never holds nodes it
  // does not upload
  bool synth = false;
  uint64_t syn_seed = 0, syn_key = 0;
  int32_t syn_mode = 0;
  double syn_scale = 0;
};

enum TaskKind : int8_t { TASK_GEMM = 0, TASK_DOT = 1, TASK_TRACE = 2 };

struct TensorRec {
  int32_t rank = 0;                  // 0 = per-slice scalar
  int32_t dim[kMaxRank] = {0, 0, 0, 0};
  int64_t slice_elems = 1;
  int32_t node = -1;                 // >= 0: an input hadron node
  int32_t task = -1;                 // >= 0: produced by this task
  int32_t level = 0;                 // 0 for nodes, 1 + max(operand levels) for task outputs
  int32_t scalar_slot = -1;          // rank 0: row of the scalar table
  int64_t bytes(int32_t Lt) const { return slice_elems * (int64_t)Lt * 16; }
};

// One unique pairwise contraction.  out[legs] = Σ_k a[...] b[...] with the contracted leg
// pairs (pa[i], pb[i]) sorted by pa; result legs = a's free legs in order, then b's
// (SURVEY.md §8(c) #9).  TRACE: a is a meson, out = Σ_i a[i][i].
struct TaskRec {
  TaskKind kind = TASK_GEMM;
  int32_t a = -1, b = -1;
  int8_t c = 0;
  int8_t pa[kMaxRank] = {0, 0, 0, 0}, pb[kMaxRank] = {0, 0, 0, 0};
  int32_t out = -1;
  int32_t level = 0;
  double flops = 0;                  // 8 real flops per complex MAC, all Lt slices
  int32_t uses = 0;                  // consumers (task operands + graph scalars)
};

struct TaskKey {
  int32_t a, b;
  int8_t c;
  int8_t pa[kMaxRank], pb[kMaxRank];
  bool operator==(const TaskKey &o) const {
    return a == o.a && b == o.b && c == o.c && std::memcmp(pa, o.pa, sizeof pa) == 0 &&
           std::memcmp(pb, o.pb, sizeof pb) == 0;
  }
};
struct TaskKeyHash {
  size_t operator()(const TaskKey &k) const {
    uint64_t h = 1469598103934665603ULL;
    auto mix = [&](uint64_t x) { h = (h ^ x) * 1099511628211ULL; };
    mix((uint32_t)k.a); mix((uint32_t)k.b); mix((uint8_t)k.c);
    for (int i = 0; i < kMaxRank; ++i) { mix((uint8_t)k.pa[i]); mix((uint8_t)k.pb[i]); }
    return (size_t)h;
  }
};

struct GraphRec {
  double coef_re = 1, coef_im = 0;
  int32_t comp_begin = 0, comp_end = 0;  // range in Context::graph_scalars
  double flops_no_dedup = 0;
};

struct SynthKey {
  uint64_t seed, key;
  int32_t mode, rank, N;
  double scale;
  bool operator==(const SynthKey &o) const {
    return seed == o.seed && key == o.key && mode == o.mode && rank == o.rank && N == o.N &&
           std::memcmp(&scale, &o.scale, sizeof scale) == 0;
  }
};
struct SynthKeyHash {
  size_t operator()(const SynthKey &k) const {
    uint64_t s;
    std::memcpy(&s, &k.scale, 8);
    return (size_t)((k.seed * 0x9E3779B97F4A7C15ULL) ^ (k.key * 0xC2B2AE3D27D4EB4FULL) ^
                    ((uint64_t)k.mode << 7) ^ ((uint64_t)k.rank << 13) ^ ((uint64_t)k.N << 17) ^ s);
  }
};

// Pinned host memory for node tensors and spills: 1 GiB chunks (cudaHostAlloc when a CUDA
// device is present, else page-aligned malloc so the host-only paths work without a GPU).
class HostArena {
 public:
  ~HostArena();
  double *alloc(int64_t bytes);
  bool pinned() const { return pinned_; }
  void release_all();
  void rewind();  // forget all allocations but keep the pinned chunks for reuse
 private:
  struct Chunk { char *base; int64_t size, used; bool pinned; };
  std::vector<Chunk> chunks_;
  struct Big { char *base; int64_t size; bool pinned; };
  std::vector<Big> big_;                  // blocks larger than a chunk, in use this round
  std::multimap<int64_t, Big> big_free_;  // kept across rewind(), reused by size
  size_t cur_ = 0;  // chunk being filled
  bool pinned_ = true;
};

class Executor;  // executor.cu

struct Plan;     // planner.cpp

struct Context {
  micco_options opt{};
  std::string last_error;
  bool sticky = false;
  int32_t Lt = -1;
  HostArena arena;
  std::vector<NodeRec> nodes;
  std::unordered_multimap<uint64_t, int32_t> node_by_hash;
  std::unordered_map<SynthKey, int32_t, SynthKeyHash> node_by_synth;
  std::vector<TensorRec> tensors;
  std::vector<TaskRec> tasks;
  std::unordered_map<TaskKey, int32_t, TaskKeyHash> task_by_key;
  std::vector<GraphRec> graphs;
  std::vector<int32_t> graph_scalars;  // tensor ids (rank 0), grouped per graph
  int64_t dedup_hits = 0;
  // canonical sub-network key of a connected component → (its scalar tensor, no-dedup flops)
  std::unordered_map<std::string, std::pair<int32_t, double>> component_by_key;
  int64_t component_dedup_hits = 0;
  int32_t n_scalar_slots = 0;
  // results of the last execute
  bool have_result = false;
  std::vector<double> corr;        // 2 * Lt
  std::vector<double> graph_vals;  // 2 * G * Lt, filled lazily
  bool graph_vals_valid = false;
  micco_stats stats{};
  std::unique_ptr<Executor> exec;
  uint8_t nccl_id[128] = {0};
  bool have_nccl_id = false;
  Context();
  ~Context();
};

// api.cpp: generate (in parallel, into pinned memory) the data of synthetic nodes not yet
// materialised
void materialize_nodes(Context &ctx, const std::vector<int32_t> &node_ids);

// builder.cpp
int32_t add_node_tensor(Context &ctx, int32_t node);
void build_graph(Context &ctx, int32_t n_inst, const int64_t *node_ids, int32_t n_edges,
                 const micco_edge *edges, const int32_t *order, double cre, double cim);
uint64_t content_hash(const double *data, int64_t n_doubles);

// planner.cpp
struct PlanOp {
  enum Kind : uint8_t { H2D = 0, P2P = 1, SPILL = 2, FREE = 3, COMPUTE = 4, FLUSH = 5 };
  Kind kind;
  int32_t gpu;     // GPU that executes the op (P2P: destination)
  int32_t src;     // P2P: source GPU
  int32_t id;      // tensor (H2D/P2P/SPILL/FREE) or task (COMPUTE)
};

struct Plan {
  int32_t n_gpus = 1;
  int32_t window_graphs = 0;
  int32_t reuse_bound[3] = {0, 0, 0};
  std::vector<PlanOp> ops;
  std::vector<int32_t> task_gpu;
  std::vector<int64_t> gpu_peak_bytes;
  int64_t bytes_h2d = 0, bytes_p2p = 0, bytes_d2h = 0, evictions = 0, cache_hits = 0;
  int64_t n_stages = 0;
  double flops = 0, max_over_mean_load = 1, predicted_s = 0;
  double predicted_overlap_s = 0;  // the same with copies overlapped: Σ_stage max_g max(flops, host, peer)
  std::vector<double> gpu_flops;
  std::vector<std::pair<int32_t, uint64_t>> final_nodes;  // (node tensor, GPU mask) left cached
  std::vector<int32_t> fused_dot;  // GEMM task → DOT task fused into its epilogue, or -1
  int64_t n_fused = 0;
  std::vector<double> stage_features;  // kBoundFeatures per stage (planner.cpp stage_features)
  std::vector<int32_t> stage_bounds;   // reuse bounds used per stage (3 each)
};

// Per-vector features of the reuse-bound model (vector size, tensor size,
// distribution, repeated rate), computed at the start of each stage:
//   0 balanceNum = ceil(pairs / n_gpus)      1 log2(mean operand bytes)
//   2 repeated rate (operand slots whose tensor occurs twice or more in the vector)
//   3 resident rate (operand slots already resident on some GPU: the locality a Gaussian
//     selection gives, L314)                  4 n_gpus
//   5 memory pressure max_g resident / budget
constexpr int kBoundFeatures = 6;
// bound_mode: how each stage's reuse bounds are chosen
enum { BOUNDS_FIXED = 0, BOUNDS_STAGE_SWEEP = 1, BOUNDS_REGRESSION = 2 };
void predict_bounds(const double *features, int32_t out[3]);  // bounds_model.cpp
void predict_bounds_raw(const double *features, double out[3]);

// Op stream from a planner thread to the executor (executor.cu): make_plan publishes the
// fused-dot table before its first stage and every stage's ops once they are final, so the
// executor enqueues stage s while stage s+1 is being planned and the GPU does not wait for
// the whole plan (every rank plans the whole DAG, so planning grows with the GPU count).
struct PlanStream {
  std::mutex m;
  std::condition_variable cv;
  std::vector<PlanOp> q;           // published, not yet taken by the executor
  std::vector<int32_t> fused_dot;  // valid once have_fused
  bool have_fused = false, done = false;
  size_t published = 0;            // plan.ops already copied into q (planner side)
  void publish_fused(const std::vector<int32_t> &f) {
    std::lock_guard<std::mutex> lk(m);
    fused_dot = f;
    have_fused = true;
    cv.notify_all();
  }
  void publish_ops(const std::vector<PlanOp> &ops) {
    if (ops.size() == published) return;
    std::lock_guard<std::mutex> lk(m);
    q.insert(q.end(), ops.begin() + (long)published, ops.end());
    published = ops.size();
    cv.notify_all();
  }
  void finish() {
    std::lock_guard<std::mutex> lk(m);
    done = true;
    have_fused = true;
    cv.notify_all();
  }
};

// The planner's cost model (bound sweep, window choice, per-vector labels), calibrated on the
// B200 (round 2): the TMA GEMM's algorithmic rate on C3 shapes (bench r02: 42.9 TFLOP/s), the
// pinned H2D copy (55.5 GB/s, profiles/fp64_peak_r01.txt probe), the NVLink peer copy per
// direction (770 GB/s, B200_PROFILING.md), and a device-local copy between logical GPUs that
// share one device (half the measured 6550 GB/s copy bandwidth: every byte is read and written).
constexpr double kModelFlopsPerS = 42.9e12;
constexpr double kModelHostGBs = 55.5;
constexpr double kModelPeerGBs = 770.0;
constexpr double kModelLocalCopyGBs = 3275.0;

struct PlanInput {
  PlanStream *stream = nullptr;                     // optional: publish ops as stages complete
  int32_t n_gpus;
  int32_t policy;
  int32_t reuse_bound[3];
  std::vector<int64_t> budget;                      // per GPU
  int32_t window_graphs;
  bool keep_inputs;
  bool fuse = true;                                 // fuse GEMM → final dot when legal
  std::vector<std::vector<int32_t>> initial_nodes;  // per GPU: node tensors already resident
  double peer_gbs, host_gbs, flops_per_s;           // cost model of the bound sweep
  int32_t bound_mode = BOUNDS_FIXED;                // per-stage bounds (BOUNDS_*)
};

Plan make_plan(const Context &ctx, const PlanInput &in);
Plan make_plan_auto(const Context &ctx, PlanInput in);  // sweeps reuse bounds when asked
// window_graphs when options.window_graphs == 0: the largest window the budget allows
// without extra host traffic (planner.cpp)
int32_t choose_window(const Context &ctx, PlanInput in);

}  // namespace micco
