// api.cpp — the C-ABI boundary (include/micco.h): argument checking, error mapping, node
// ingest (pinned copy + content-hash dedup), and dispatch to the
// builder / planner / executor.  No computation on the hot path happens here.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdlib>
#include <cstring>
#include <thread>

#include "core.h"
#include "executor.h"
#include "kernels.h"
#include "micco_inputs/synth.h"
#include "scheduler.h"

namespace micco {

[[noreturn]] void fail(micco_status code, const std::string &msg) { throw Error{code, msg}; }

Context::Context() = default;
Context::~Context() = default;

HostArena::~HostArena() { release_all(); }

void HostArena::release_all() {
  for (auto &c : chunks_) {
    if (c.pinned) cudaFreeHost(c.base); else std::free(c.base);
  }
  chunks_.clear();
  cur_ = 0;
  rewind();
  for (auto &kv : big_free_) {
    if (kv.second.pinned) cudaFreeHost(kv.second.base); else std::free(kv.second.base);
  }
  big_free_.clear();
}

void HostArena::rewind() {
  for (auto &c : chunks_) c.used = 0;
  cur_ = 0;
  // large blocks go back to a free list: pinning gigabytes costs ~0.5 s/GB, so an execute that
  // spills rank-4 intermediates would otherwise re-pin them every time
  for (auto &b : big_) big_free_.emplace(b.size, b);
  big_.clear();
}

double *HostArena::alloc(int64_t bytes) {
  constexpr int64_t kChunk = 1LL << 30;
  bytes = (bytes + 255) & ~int64_t(255);
  auto raw = [&](int64_t n, bool &pinned) -> char * {
    void *p = nullptr;
    if (pinned_ && cudaHostAlloc(&p, (size_t)n, cudaHostAllocPortable) == cudaSuccess) {
      pinned = true;
      return (char *)p;
    }
    cudaGetLastError();
    pinned_ = false;  // no CUDA device: plain memory (host-only paths; execute will fail loudly)
    pinned = false;
    if (posix_memalign(&p, 4096, (size_t)n) != 0) return nullptr;
    return (char *)p;
  };
  if (bytes > kChunk / 4) {
    auto it = big_free_.lower_bound(bytes);  // smallest kept block that fits, if not wasteful
    if (it != big_free_.end() && it->first <= bytes + bytes / 4) {
      Big b = it->second;
      big_free_.erase(it);
      big_.push_back(b);
      return (double *)b.base;
    }
    bool pinned;
    char *p = raw(bytes, pinned);
    if (!p) fail(MICCO_ERR_OOM, "host allocation failed");
    big_.push_back({p, bytes, pinned});
    return (double *)p;
  }
  while (cur_ < chunks_.size() && chunks_[cur_].used + bytes > chunks_[cur_].size) ++cur_;
  if (cur_ == chunks_.size()) {
    bool pinned;
    char *p = raw(kChunk, pinned);
    if (!p) fail(MICCO_ERR_OOM, "host allocation failed");
    chunks_.push_back({p, kChunk, 0, pinned});
  }
  Chunk &c = chunks_[cur_];
  char *p = c.base + c.used;
  c.used += bytes;
  return (double *)p;
}

}  // namespace micco

using namespace micco;

struct micco_ctx {
  Context c;
};

namespace {

template <typename F>
micco_status guard(micco_ctx *ctx, F &&f) {
  if (!ctx) return MICCO_ERR_ARG;
  if (ctx->c.sticky) {
    ctx->c.last_error = "context is unusable after an earlier CUDA/NCCL failure: " + ctx->c.last_error;
    return MICCO_ERR_STATE;
  }
  try {
    f();
    ctx->c.last_error.clear();
    return MICCO_OK;
  } catch (const Error &e) {
    ctx->c.last_error = e.msg;
    if (e.code == MICCO_ERR_CUDA || e.code == MICCO_ERR_NCCL) ctx->c.sticky = true;
    return e.code;
  } catch (const std::bad_alloc &) {
    ctx->c.last_error = "host out of memory";
    return MICCO_ERR_OOM;
  } catch (...) {
    ctx->c.last_error = "internal error";
    return MICCO_ERR_STATE;
  }
}

void check_lt(Context &c, int32_t Lt) {
  if (Lt < 1) fail(MICCO_ERR_ARG, "Lt must be >= 1");
  if (c.Lt < 0) c.Lt = Lt;
  else if (c.Lt != Lt) fail(MICCO_ERR_ARG, "Lt differs from earlier nodes");
}

void check_shape(int32_t rank, int32_t N) {
  if (rank != 2 && rank != 3) fail(MICCO_ERR_ARG, "rank must be 2 (meson) or 3 (baryon)");
  if (N < 1 || N > 65536) fail(MICCO_ERR_ARG, "N out of range");
}

int32_t new_node(Context &c, int32_t rank, int32_t N, bool allocate = true) {
  NodeRec nd;
  nd.rank = rank;
  nd.N = N;
  nd.slice_elems = 1;
  for (int i = 0; i < rank; ++i) nd.slice_elems *= N;
  if (allocate) nd.host = c.arena.alloc(nd.slice_elems * (int64_t)c.Lt * 16);
  c.nodes.push_back(nd);
  int32_t id = (int32_t)c.nodes.size() - 1;
  c.nodes[id].tensor = add_node_tensor(c, id);
  return id;
}

}  // namespace

extern "C" {

MICCO_API void micco_options_default(micco_options *opt) {
  if (!opt) return;
  std::memset(opt, 0, sizeof(*opt));
  opt->struct_size = sizeof(micco_options);
  opt->policy = MICCO_POLICY_MICCO;
  opt->deterministic = 1;
}

MICCO_API micco_status micco_create(micco_ctx **out, const micco_options *opt) {
  if (!out) return MICCO_ERR_ARG;
  *out = nullptr;
  micco_options o;
  micco_options_default(&o);
  if (opt) {
    if (opt->struct_size < offsetof(micco_options, keep_inputs_resident)) return MICCO_ERR_ARG;
    std::memcpy(&o, opt, std::min(opt->struct_size, sizeof(o)));
    o.struct_size = sizeof(o);
  }
  if (o.policy < 0 || o.policy > 4 || o.window_graphs < 0 || o.mem_budget_bytes < 0 || o.dist_world < 0 ||
      o.reorder < 0 || o.reorder > 1 || o.bound_model < 0 || o.bound_model > 2 ||
      o.scalar_tables < 0 || o.scalar_tables > 1 ||
      (o.dist_world > 0 && (o.dist_rank < 0 || o.dist_rank >= o.dist_world)))
    return MICCO_ERR_ARG;
  micco_ctx *c = new (std::nothrow) micco_ctx;
  if (!c) return MICCO_ERR_OOM;
  c->c.opt = o;
  *out = c;
  return MICCO_OK;
}

MICCO_API void micco_destroy(micco_ctx *ctx) {
  if (!ctx) return;
  ctx->c.exec.reset();
  delete ctx;
}

MICCO_API micco_status micco_add_hadron_node(micco_ctx *ctx, int32_t rank, int32_t N, int32_t Lt,
                                             const double *data, int64_t *node_id) {
  return guard(ctx, [&] {
    Context &c = ctx->c;
    if (!data || !node_id) fail(MICCO_ERR_ARG, "add_hadron_node: null pointer");
    check_shape(rank, N);
    check_lt(c, Lt);
    int64_t elems = 1;
    for (int i = 0; i < rank; ++i) elems *= N;
    const int64_t nd = 2 * elems * (int64_t)Lt;
    const uint64_t h = content_hash(data, nd);
    auto range = c.node_by_hash.equal_range(h);
    for (auto it = range.first; it != range.second; ++it) {
      const NodeRec &o = c.nodes[it->second];
      if (o.rank == rank && o.N == N && std::memcmp(o.host, data, (size_t)nd * 8) == 0) {
        *node_id = it->second;
        return;
      }
    }
    int32_t id = new_node(c, rank, N);
    std::memcpy(c.nodes[id].host, data, (size_t)nd * 8);
    c.nodes[id].hash = h;
    c.node_by_hash.emplace(h, id);
    *node_id = id;
  });
}

MICCO_API micco_status micco_add_hadron_nodes_synth(micco_ctx *ctx, int32_t count, int32_t rank, int32_t N,
                                                    int32_t Lt, uint64_t seed, const uint64_t *keys,
                                                    int32_t mode, double scale, int64_t *node_ids) {
  return guard(ctx, [&] {
    Context &c = ctx->c;
    if (count < 0 || (count > 0 && (!keys || !node_ids))) fail(MICCO_ERR_ARG, "add_hadron_nodes_synth: bad args");
    if (mode != MICCO_SYNTH_UNIFORM && mode != MICCO_SYNTH_INT3) fail(MICCO_ERR_ARG, "bad synth mode");
    check_shape(rank, N);
    check_lt(c, Lt);
    const bool lazy = c.opt.dist_world > 0;  // multi-process: generate on first use by this rank
    std::vector<int32_t> todo;
    for (int32_t i = 0; i < count; ++i) {
      SynthKey k{seed, keys[i], mode, rank, N, scale};
      auto it = c.node_by_synth.find(k);
      if (it != c.node_by_synth.end()) { node_ids[i] = it->second; continue; }
      int32_t id = new_node(c, rank, N, /*allocate=*/false);
      NodeRec &nd = c.nodes[id];
      nd.synth = true;
      nd.syn_seed = seed;
      nd.syn_key = keys[i];
      nd.syn_mode = mode;
      nd.syn_scale = scale;
      c.node_by_synth.emplace(k, id);
      todo.push_back(id);
      node_ids[i] = id;
    }
    if (!lazy) materialize_nodes(c, todo);
  });
}

}  // extern "C"

namespace micco {

void materialize_nodes(Context &c, const std::vector<int32_t> &node_ids) {
  std::vector<int32_t> todo;
  for (int32_t id : node_ids)
    if (c.nodes[id].synth && !c.nodes[id].host) todo.push_back(id);
  if (todo.empty()) return;
  for (int32_t id : todo) c.nodes[id].host = c.arena.alloc(c.nodes[id].slice_elems * (int64_t)c.Lt * 16);
  // split every node into blocks so all host threads stay busy
  const int64_t blk = 1 << 18;
  std::vector<int64_t> first_block(todo.size() + 1, 0);
  for (size_t i = 0; i < todo.size(); ++i) {
    const int64_t per = c.nodes[todo[i]].slice_elems * (int64_t)c.Lt;
    first_block[i + 1] = first_block[i] + (per + blk - 1) / blk;
  }
  const int64_t total = first_block.back();
  unsigned nt = std::max(1u, std::min(64u, std::thread::hardware_concurrency()));
  std::vector<std::thread> th;
  std::atomic<int64_t> next{0};
  for (unsigned w = 0; w < nt; ++w)
    th.emplace_back([&] {
      for (int64_t b; (b = next.fetch_add(1)) < total;) {
        const size_t i = std::upper_bound(first_block.begin(), first_block.end(), b) - first_block.begin() - 1;
        const NodeRec &nd = c.nodes[todo[i]];
        const int64_t per = nd.slice_elems * (int64_t)c.Lt;
        const int64_t first = (b - first_block[i]) * blk;
        const int64_t cnt = std::min(blk, per - first);
        micco_synth_fill(nd.host + 2 * first, nd.syn_seed, nd.syn_key, first, cnt, nd.syn_mode, nd.syn_scale);
      }
    });
  for (auto &t : th) t.join();
}

}  // namespace micco

extern "C" {

MICCO_API micco_status micco_add_graph(micco_ctx *ctx, int32_t n_inst, const int64_t *node_ids, int32_t n_edges,
                                       const micco_edge *edges, const int32_t *order, double coef_re,
                                       double coef_im, int64_t *graph_id) {
  return guard(ctx, [&] {
    Context &c = ctx->c;
    build_graph(c, n_inst, node_ids, n_edges, edges, order, coef_re, coef_im);
    if (graph_id) *graph_id = (int64_t)c.graphs.size() - 1;
  });
}

MICCO_API micco_status micco_execute(micco_ctx *ctx, int32_t n_gpus, const int32_t *reuse_bound) {
  return guard(ctx, [&] {
    Context &c = ctx->c;
    if (n_gpus < 1 || n_gpus > 64) fail(MICCO_ERR_ARG, "n_gpus must be in [1, 64]");
    if (c.graphs.empty()) fail(MICCO_ERR_STATE, "execute: no graphs");
    if (reuse_bound)
      for (int i = 0; i < 3; ++i)
        if (reuse_bound[i] < 0) fail(MICCO_ERR_ARG, "reuse bounds must be >= 0");
    if (c.opt.dist_world > 0 && n_gpus != c.opt.dist_world)
      fail(MICCO_ERR_ARG, "multi-process mode: n_gpus must equal the world size");
    if (!c.exec) c.exec.reset(new Executor(c));
    c.have_result = false;
    c.graph_vals_valid = false;
    c.exec->execute(n_gpus, reuse_bound);
    c.have_result = true;
  });
}

namespace {
Plan host_plan(Context &c, int32_t n_gpus, const int32_t *reuse_bound, int32_t bound_mode = -1) {
  if (n_gpus < 1 || n_gpus > 64) fail(MICCO_ERR_ARG, "n_gpus must be in [1, 64]");
  if (c.opt.mem_budget_bytes <= 0) fail(MICCO_ERR_ARG, "micco_plan needs options.mem_budget_bytes");
  PlanInput in;
  in.n_gpus = n_gpus;
  in.policy = c.opt.policy;
  for (int i = 0; i < 3; ++i) in.reuse_bound[i] = reuse_bound ? reuse_bound[i] : 0;
  in.budget.assign(n_gpus, c.opt.mem_budget_bytes);
  in.window_graphs = c.opt.window_graphs;
  in.keep_inputs = c.opt.keep_inputs_resident != 0;
  in.peer_gbs = kModelPeerGBs;  // (host-only plans model a multi-GPU node)
  in.host_gbs = kModelHostGBs;
  in.flops_per_s = kModelFlopsPerS;
  if (bound_mode < 0) bound_mode = reuse_bound ? BOUNDS_FIXED : c.opt.bound_model;
  if (bound_mode != BOUNDS_FIXED) in.bound_mode = bound_mode;
  in.window_graphs = choose_window(c, in);
  const char *warm = getenv("MICCO_PLAN_WARM");  // tools: plan a repeat execute (keep_inputs
  if (warm && warm[0] == '1' && in.keep_inputs) {  // replicas left by a first, cold one)
    Plan cold = reuse_bound || bound_mode != BOUNDS_FIXED ? make_plan(c, in) : make_plan_auto(c, in);
    in.initial_nodes.assign(n_gpus, {});
    for (const auto &fn : cold.final_nodes)
      for (int g = 0; g < n_gpus; ++g)
        if ((fn.second >> g) & 1) in.initial_nodes[g].push_back(fn.first);
    if (!reuse_bound && bound_mode == BOUNDS_FIXED)
      for (int i = 0; i < 3; ++i) in.reuse_bound[i] = cold.reuse_bound[i];
    return make_plan(c, in);
  }
  if (bound_mode != BOUNDS_FIXED) {
    in.bound_mode = bound_mode;
    return make_plan(c, in);
  }
  return reuse_bound ? make_plan(c, in) : make_plan_auto(c, in);
}
}  // namespace

MICCO_API micco_status micco_plan_stages(micco_ctx *ctx, int32_t n_gpus, int32_t bound_mode,
                                         const int32_t *reuse_bound, int64_t max_stages, double *features,
                                         int32_t *bounds, int64_t *n_stages, double *predicted_s) {
  return guard(ctx, [&] {
    if (bound_mode < 0 || bound_mode > 2) fail(MICCO_ERR_ARG, "bound_mode must be 0, 1 or 2");
    Plan p = host_plan(ctx->c, n_gpus, reuse_bound, bound_mode);
    const int64_t ns = (int64_t)p.stage_bounds.size() / 3;
    if (n_stages) *n_stages = ns;
    if (predicted_s) *predicted_s = p.predicted_s;
    const int64_t k = std::min(max_stages, ns);
    if (features) std::copy(p.stage_features.begin(), p.stage_features.begin() + k * kBoundFeatures, features);
    if (bounds) std::copy(p.stage_bounds.begin(), p.stage_bounds.begin() + k * 3, bounds);
  });
}

MICCO_API void micco_predict_bounds(const double *features, double *raw, int32_t *bounds) {
  if (!features) return;
  int32_t b[3];
  double r[3];
  predict_bounds_raw(features, r);
  predict_bounds(features, b);
  for (int i = 0; i < 3; ++i) {
    if (raw) raw[i] = r[i];
    if (bounds) bounds[i] = b[i];
  }
}

MICCO_API micco_status micco_plan_ops(micco_ctx *ctx, int32_t n_gpus, const int32_t *reuse_bound, int64_t max_ops,
                                      int32_t *ops, int64_t *n_ops, int32_t *fused) {
  return guard(ctx, [&] {
    Plan p = host_plan(ctx->c, n_gpus, reuse_bound);
    if (n_ops) *n_ops = (int64_t)p.ops.size();
    if (ops)
      for (int64_t i = 0; i < std::min<int64_t>(max_ops, (int64_t)p.ops.size()); ++i) {
        ops[4 * i] = p.ops[i].kind;
        ops[4 * i + 1] = p.ops[i].gpu;
        ops[4 * i + 2] = p.ops[i].src;
        ops[4 * i + 3] = p.ops[i].id;
      }
    if (fused) std::copy(p.fused_dot.begin(), p.fused_dot.end(), fused);
  });
}

MICCO_API micco_status micco_dag(const micco_ctx *ctx, int64_t *n_tensors, int64_t *n_tasks, int64_t *tensor_bytes,
                                 int32_t *tensor_task, int32_t *task_info) {
  if (!ctx) return MICCO_ERR_ARG;
  const Context &c = ctx->c;
  if (n_tensors) *n_tensors = (int64_t)c.tensors.size();
  if (n_tasks) *n_tasks = (int64_t)c.tasks.size();
  for (size_t x = 0; x < c.tensors.size(); ++x) {
    if (tensor_bytes) tensor_bytes[x] = c.tensors[x].rank > 0 ? c.tensors[x].bytes(c.Lt) : 0;
    if (tensor_task) tensor_task[x] = c.tensors[x].task;
  }
  if (task_info)
    for (size_t t = 0; t < c.tasks.size(); ++t) {
      task_info[4 * t] = c.tasks[t].kind;
      task_info[4 * t + 1] = c.tasks[t].a;
      task_info[4 * t + 2] = c.tasks[t].b;
      task_info[4 * t + 3] = c.tasks[t].out;
    }
  return MICCO_OK;
}

MICCO_API micco_status micco_plan(micco_ctx *ctx, int32_t n_gpus, const int32_t *reuse_bound, micco_stats *out,
                                  int32_t *assign) {
  return guard(ctx, [&] {
    Context &c = ctx->c;
    Plan p = host_plan(c, n_gpus, reuse_bound);
    if (out) {
      micco_stats s{};
      s.struct_size = sizeof(s);
      s.unique_tasks = (int64_t)c.tasks.size();
      s.dedup_hits = c.dedup_hits;
      s.component_dedup_hits = c.component_dedup_hits;
      for (const TaskRec &t : c.tasks) (t.kind == TASK_GEMM ? s.n_gemm : s.n_dot)++;
      s.model_s = p.predicted_s;
      for (int64_t b : p.gpu_peak_bytes) s.peak_bytes = std::max(s.peak_bytes, b);
      s.window_graphs = p.window_graphs;
      s.model_overlap_s = p.predicted_overlap_s;
      s.n_stages = p.n_stages;
      s.bytes_h2d = p.bytes_h2d;
      s.bytes_p2p = p.bytes_p2p;
      s.bytes_d2h = p.bytes_d2h;
      s.evictions = p.evictions;
      s.cache_hits = p.cache_hits;
      s.flops = p.flops;
      for (const GraphRec &g : c.graphs) s.flops_no_dedup += g.flops_no_dedup;
      s.max_over_mean_load = p.max_over_mean_load;
      for (int i = 0; i < 3; ++i) s.reuse_bound[i] = p.reuse_bound[i];
      s.n_gpus = n_gpus;
      size_t n = std::min(out->struct_size ? out->struct_size : sizeof(s), sizeof(s));
      std::memcpy(out, &s, n);
    }
    if (assign) std::copy(p.task_gpu.begin(), p.task_gpu.end(), assign);
  });
}

MICCO_API micco_status micco_get_correlator(const micco_ctx *ctx, int32_t t, double out[2]) {
  if (!ctx || !out) return MICCO_ERR_ARG;
  const Context &c = ctx->c;
  if (!c.have_result) return MICCO_ERR_STATE;
  if (t < 0 || t >= c.Lt) return MICCO_ERR_RANGE;
  out[0] = c.corr[2 * t];
  out[1] = c.corr[2 * t + 1];
  return MICCO_OK;
}

MICCO_API micco_status micco_get_graph_value(const micco_ctx *ctx, int64_t graph_id, int32_t t, double out[2]) {
  if (!ctx || !out) return MICCO_ERR_ARG;
  micco_ctx *m = const_cast<micco_ctx *>(ctx);
  Context &c = m->c;
  if (!c.have_result) return MICCO_ERR_STATE;
  if (t < 0 || t >= c.Lt || graph_id < 0 || graph_id >= (int64_t)c.graphs.size()) return MICCO_ERR_RANGE;
  if (!c.graph_vals_valid) {
    micco_status st = guard(m, [&] { c.exec->fetch_graph_values(); });
    if (st != MICCO_OK) return st;
  }
  out[0] = c.graph_vals[2 * (graph_id * c.Lt + t)];
  out[1] = c.graph_vals[2 * (graph_id * c.Lt + t) + 1];
  return MICCO_OK;
}

MICCO_API const char *micco_last_error(const micco_ctx *ctx) {
  if (!ctx) return "null context";
  return ctx->c.last_error.c_str();
}

MICCO_API micco_status micco_get_stats(const micco_ctx *ctx, micco_stats *out) {
  if (!ctx || !out || out->struct_size == 0) return MICCO_ERR_ARG;
  size_t n = std::min(out->struct_size, sizeof(micco_stats));
  micco_stats s = ctx->c.stats;
  s.struct_size = n;
  std::memcpy(out, &s, n);
  return MICCO_OK;
}

MICCO_API micco_status micco_probe_fp64_peak(double seconds, double *burst_tflops, double *sustained_tflops) {
  if (!burst_tflops || !sustained_tflops || !(seconds >= 0)) return MICCO_ERR_ARG;
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess || n < 1) return MICCO_ERR_CUDA;
  return micco::probe_fp64_peak(seconds, burst_tflops, sustained_tflops) == cudaSuccess ? MICCO_OK : MICCO_ERR_CUDA;
}

MICCO_API micco_status micco_release_cache(micco_ctx *ctx) {
  return guard(ctx, [&] {
    if (ctx->c.exec) ctx->c.exec->release_cache();
  });
}

MICCO_API micco_status micco_set_policy(micco_ctx *ctx, int32_t policy) {
  return guard(ctx, [&] {
    if (policy < 0 || policy > 4) fail(MICCO_ERR_ARG, "unknown policy");
    if (ctx->c.exec) ctx->c.exec->release_cache();
    ctx->c.opt.policy = policy;
  });
}

MICCO_API micco_status micco_nccl_unique_id(uint8_t out[128]) {
  if (!out) return MICCO_ERR_ARG;
  return nccl_unique_id(out);
}

MICCO_API micco_status micco_set_nccl_id(micco_ctx *ctx, const uint8_t id[128]) {
  return guard(ctx, [&] {
    if (!id) fail(MICCO_ERR_ARG, "null id");
    std::memcpy(ctx->c.nccl_id, id, 128);
    ctx->c.have_nccl_id = true;
  });
}

MICCO_API micco_status micco_debug_schedule(int32_t n_gpus, const int32_t reuse_bound[3], double gpu_max_memory,
                                            int32_t n_vectors, const int64_t *vec_off, const double *pairs,
                                            int32_t n_resident, const int64_t *resident, int32_t *out_gpu) {
  if (n_gpus < 1 || n_gpus > 64 || !reuse_bound || n_vectors < 0 || (n_vectors > 0 && (!vec_off || !pairs || !out_gpu)) ||
      n_resident < 0 || (n_resident > 0 && !resident))
    return MICCO_ERR_ARG;
  // the oracle's model (oracle/sched.py): residency only grows, mapGPUMem counts every tensor
  // once per GPU it lands on, no eviction
  std::unordered_map<int64_t, uint64_t> mask;
  Scheduler s(n_gpus, MICCO_POLICY_MICCO, reuse_bound,
              std::vector<int64_t>(n_gpus, gpu_max_memory >= 9e18 ? INT64_MAX : (int64_t)gpu_max_memory));
  for (int32_t i = 0; i < n_resident; ++i) {
    int64_t t = resident[2 * i], g = resident[2 * i + 1];
    if (g < 0 || g >= n_gpus) return MICCO_ERR_ARG;
    mask[t] |= 1ULL << g;
  }
  for (int32_t v = 0; v < n_vectors; ++v) {
    s.begin_vector(vec_off[v + 1] - vec_off[v]);
    for (int64_t i = vec_off[v]; i < vec_off[v + 1]; ++i) {
      const double *p = pairs + 7 * i;
      int64_t t1 = (int64_t)p[0], t2 = (int64_t)p[1], to = (int64_t)p[2];
      SchedPair sp;
      sp.m1 = mask[t1];
      sp.m2 = mask[t2];
      sp.same = t1 == t2;
      sp.flops = p[3];
      sp.b1 = (int64_t)p[4];
      sp.b2 = sp.same ? 0 : (int64_t)p[5];
      sp.bout = (int64_t)p[6];
      int g = s.decide(sp);
      out_gpu[i] = g;
      const uint64_t bit = 1ULL << g;
      if (!(mask[t1] & bit)) { mask[t1] |= bit; s.mem[g] += sp.b1; }
      if (!sp.same && !(mask[t2] & bit)) { mask[t2] |= bit; s.mem[g] += sp.b2; }
      mask[to] |= bit;
      s.mem[g] += sp.bout;
      s.account(g, sp);
    }
  }
  return MICCO_OK;
}

}  // extern "C"
