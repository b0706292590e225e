// planner.cpp — turns the task DAG into per-GPU operation streams.
//
//  * Stages (Fig. 1 L48): graphs are taken in windows (a stream of vectors,
//    Fig. 6); inside a window a task's stage is its DAG level, so the pairs of one
//    stage are independent and stages run in order.
//  * Each pair of a stage is assigned a GPU by the scheduler (Alg. 1/2, scheduler.cpp).
//  * A per-GPU HBM cache is simulated exactly: an operand is a hit, a peer copy over
//    NVLink (P2P) or a host upload (H2D); when a GPU would exceed its budget
//    (GPUMaxMemory, L193) replicas are evicted — dead ones first, then those with another
//    copy, furthest next use first (the DAG is known, so next use is exact), then sole
//    copies are spilled to pinned host memory (SURVEY.md §8(c) reading #19; the paper is
//    silent on the victim, L199/L250).
//  * Refcounts free intermediates after their last consumer.
// The output is a flat, globally ordered op list that the executor replays; in
// multi-process mode every rank builds the identical plan.
#include <algorithm>
#include <climits>
#include <cmath>
#include <limits>
#include <cstdlib>
#include <string>

#include "core.h"
#include "layout.h"
#include "scheduler.h"

namespace micco {

namespace {

struct PlanState {
  const Context &ctx;
  const PlanInput &in;
  Plan &plan;
  int n;
  int32_t Lt;
  std::vector<uint64_t> mask;          // GPUs holding a replica
  std::vector<char> on_host;           // spilled copy on host (nodes are always on host)
  std::vector<int32_t> uses_left;
  std::vector<std::vector<int32_t>> use_stages;  // sorted stage ids where the tensor is an operand
  std::vector<std::vector<int32_t>> res;         // resident tensors per GPU
  std::vector<std::vector<int32_t>> res_pos;     // index in res[g], -1 if absent
  std::vector<std::vector<int32_t>> pin;         // pin epoch per GPU per tensor
  std::vector<int32_t> epoch;
  std::vector<int64_t> mem;
  std::vector<double> st_flops, st_h2d, st_p2p, st_d2h;
  int32_t stage = 0;

  PlanState(const Context &c, const PlanInput &i, Plan &p)
      : ctx(c), in(i), plan(p), n(i.n_gpus), Lt(c.Lt) {}

  int64_t bytes(int32_t x) const { return ctx.tensors[x].bytes(Lt); }
  bool is_node(int32_t x) const { return ctx.tensors[x].node >= 0; }

  void add_res(int g, int32_t x) {
    res_pos[g][x] = (int32_t)res[g].size();
    res[g].push_back(x);
    mask[x] |= 1ULL << g;
    mem[g] += bytes(x);
    plan.gpu_peak_bytes[g] = std::max(plan.gpu_peak_bytes[g], mem[g]);
  }
  void drop_res(int g, int32_t x) {
    int32_t i = res_pos[g][x];
    int32_t last = res[g].back();
    res[g][i] = last;
    res_pos[g][last] = i;
    res[g].pop_back();
    res_pos[g][x] = -1;
    mask[x] &= ~(1ULL << g);
    mem[g] -= bytes(x);
  }
  void emit(PlanOp::Kind k, int g, int src, int32_t id) { plan.ops.push_back(PlanOp{k, g, src, id}); }

  int32_t next_use(int32_t x) const {
    const auto &u = use_stages[x];
    auto it = std::lower_bound(u.begin(), u.end(), stage);
    return it == u.end() ? std::numeric_limits<int32_t>::max() : *it;
  }

  // Evict unpinned replicas on g until need more bytes fit; false if impossible.  Dead and
  // replicated tensors (classes 0, 1: no host traffic to evict) are evicted down to a low-water
  // mark budget/64 below the need, so the scan-and-sort runs once per ~budget/64 bytes instead of
  // once per allocation (a full 8-GPU C2 plan evicts ~17k replicas: 17 s → 0.2 s of planning);
  // sole copies (class 2, a D2H spill) only to fit the need itself.
  bool make_room(int g, int64_t need) {
    const int64_t budget = in.budget[g];
    if (mem[g] + need <= budget) return true;
    const int64_t low = budget - budget / 64;
    struct Cand { int cls; int32_t next; int32_t x; };
    std::vector<Cand> cands;
    for (int32_t x : res[g]) {
      if (pin[g][x] == epoch[g]) continue;
      int cls;
      if (uses_left[x] == 0) cls = 0;
      else if (is_node(x) || on_host[x] || (mask[x] & ~(1ULL << g))) cls = 1;
      else cls = 2;
      cands.push_back({cls, next_use(x), x});
    }
    std::sort(cands.begin(), cands.end(), [](const Cand &a, const Cand &b) {
      if (a.cls != b.cls) return a.cls < b.cls;
      if (a.next != b.next) return a.next > b.next;
      return a.x < b.x;
    });
    for (const Cand &c : cands) {
      if (mem[g] + need <= (c.cls == 2 ? budget : low)) break;
      if (c.cls == 2) {  // sole copy: spill to pinned host memory first
        emit(PlanOp::SPILL, g, -1, c.x);
        on_host[c.x] = 1;
        plan.bytes_d2h += bytes(c.x);
        st_d2h[g] += (double)bytes(c.x);
      }
      emit(PlanOp::FREE, g, -1, c.x);
      drop_res(g, c.x);
      ++plan.evictions;
    }
    return mem[g] + need <= budget;
  }

  void fetch(int g, int32_t x) {
    uint64_t others = mask[x] & ~(1ULL << g);
    if (others) {  // a peer holds it: NVLink peer copy
      int src = __builtin_ctzll(others);
      emit(PlanOp::P2P, g, src, x);
      plan.bytes_p2p += bytes(x);
      st_p2p[g] += (double)bytes(x);
    } else {
      if (!is_node(x) && !on_host[x]) fail(MICCO_ERR_STATE, "planner: lost the only copy of a tensor");
      emit(PlanOp::H2D, g, -1, x);
      plan.bytes_h2d += bytes(x);
      st_h2d[g] += (double)bytes(x);
    }
    add_res(g, x);
  }

  void release(int32_t x) {  // last consumer done
    if (is_node(x) && in.keep_inputs) return;  // stays cached (dead → evicted first)
    for (uint64_t m = mask[x]; m; m &= m - 1) {
      int g = __builtin_ctzll(m);
      emit(PlanOp::FREE, g, -1, x);
      drop_res(g, x);
    }
    if (!is_node(x) && on_host[x]) {
      emit(PlanOp::FREE, -1, -1, x);  // release the host spill copy
      on_host[x] = 0;
    }
  }
};

}  // namespace

Plan make_plan(const Context &ctx, const PlanInput &in) {
  Plan plan;
  const int n = in.n_gpus;
  plan.n_gpus = n;
  for (int i = 0; i < 3; ++i) plan.reuse_bound[i] = in.reuse_bound[i];
  const int32_t T = (int32_t)ctx.tasks.size(), NT = (int32_t)ctx.tensors.size();
  const int32_t G = (int32_t)ctx.graphs.size();
  plan.task_gpu.assign(T, -1);
  plan.gpu_peak_bytes.assign(n, 0);
  plan.gpu_flops.assign(n, 0.0);

  // 1. window of every task = window of the first graph that needs it
  const int32_t W = in.window_graphs > 0 ? in.window_graphs : 256;
  plan.window_graphs = W;
  // Graphs are windowed in an order that keeps graphs sharing an intermediate together:
  // key = the smallest id among the level-1 tasks a graph depends on (its first shared
  // product), ties in graph order.  Shared intermediates then live for a few windows instead
  // of the whole stream (fewer evictions and spills).  C(t) does not depend on this order
  // (the final sum runs over graph ids in a fixed order).
  std::vector<int32_t> gorder(G);
  {
    std::vector<int32_t> key(G, INT32_MAX), first1(T, -1);
    for (int32_t t = 0; t < T; ++t) {  // smallest level-1 task reachable from each task
      const TaskRec &tk = ctx.tasks[t];  // operands precede their consumers in id order
      int32_t k = INT32_MAX;
      for (int32_t op : {tk.a, tk.b}) {
        if (op < 0) continue;
        const int32_t pt = ctx.tensors[op].task;
        if (pt >= 0) k = std::min(k, first1[pt]);
      }
      first1[t] = (k == INT32_MAX) ? t : k;
    }
    for (int32_t g = 0; g < G; ++g)
      for (int32_t c = ctx.graphs[g].comp_begin; c < ctx.graphs[g].comp_end; ++c) {
        const int32_t t0 = ctx.tensors[ctx.graph_scalars[c]].task;
        if (t0 >= 0) key[g] = std::min(key[g], first1[t0]);
      }
    for (int32_t g = 0; g < G; ++g) gorder[g] = g;
    std::stable_sort(gorder.begin(), gorder.end(), [&](int32_t x, int32_t y) { return key[x] < key[y]; });
  }
  std::vector<int32_t> task_window(T, -1);
  std::vector<int32_t> stack;
  for (int32_t gi = 0; gi < G; ++gi) {
    const int32_t g = gorder[gi];
    const int32_t w = gi / W;
    for (int32_t c = ctx.graphs[g].comp_begin; c < ctx.graphs[g].comp_end; ++c) {
      int32_t t0 = ctx.tensors[ctx.graph_scalars[c]].task;
      if (t0 >= 0 && task_window[t0] < 0) { task_window[t0] = w; stack.push_back(t0); }
      while (!stack.empty()) {
        int32_t t = stack.back();
        stack.pop_back();
        for (int32_t op : {ctx.tasks[t].a, ctx.tasks[t].b}) {
          if (op < 0) continue;
          int32_t pt = ctx.tensors[op].task;
          if (pt >= 0 && task_window[pt] < 0) { task_window[pt] = w; stack.push_back(pt); }
        }
      }
    }
  }
  // 1b. fuse a final dot into the GEMM that produces its operand when that product X is a
  // matrix used by nothing else: X is never written, the dot's other operand Y is read in
  // the GEMM epilogue (kernels.h GemmDesc::D), so the fused GEMM runs one stage after Y's
  // producer at the earliest (plevel).  Decided from the DAG alone, so it is identical for
  // every GPU count.
  std::vector<int32_t> plevel(T);
  for (int32_t t = 0; t < T; ++t) plevel[t] = ctx.tasks[t].level;
  plan.fused_dot.assign(T, -1);
  std::vector<char> skip(T, 0);
  std::vector<int32_t> extra(T, -1);  // fused GEMM task → Y
  if (in.fuse) {
    std::vector<int32_t> consumers(NT, 0);
    for (int32_t t = 0; t < T; ++t) {
      const TaskRec &tk = ctx.tasks[t];
      if (tk.a >= 0) ++consumers[tk.a];
      if (tk.b >= 0 && tk.b != tk.a) ++consumers[tk.b];
    }
    for (int32_t d = 0; d < T; ++d) {
      const TaskRec &dk = ctx.tasks[d];
      if (dk.kind != TASK_DOT || dk.a == dk.b || task_window[d] < 0) continue;
      for (int side = 0; side < 2; ++side) {
        const int32_t X = side == 0 ? dk.a : dk.b, Y = side == 0 ? dk.b : dk.a;
        const int32_t pt = ctx.tensors[X].task;
        if (pt < 0 || consumers[X] != 1 || ctx.tensors[X].rank != 2) continue;
        const TaskRec &pk = ctx.tasks[pt];
        if (pk.kind != TASK_GEMM || plan.fused_dot[pt] >= 0) continue;
        const TensorRec &A = ctx.tensors[pk.a], &B = ctx.tensors[pk.b];
        if (A.rank - pk.c != 1 || B.rank - pk.c != 1) continue;  // one M leg, one N leg
        GemmLayout L;
        if (!gemm_layout(A.rank, A.dim, B.rank, B.dim, pk.c, pk.pa, pk.pb, L) || gemm_class(L) == 4) continue;
        plan.fused_dot[pt] = d;
        extra[pt] = Y;
        plevel[pt] = std::max(plevel[pt], ctx.tensors[Y].level + 1);
        skip[d] = 1;
        ++plan.n_fused;
        break;
      }
    }
  }
  auto operands = [&](int32_t t, int32_t out[3]) {  // distinct tensors a task reads
    const TaskRec &tk = ctx.tasks[t];
    int k = 0;
    out[k++] = tk.a;
    if (tk.b >= 0 && tk.b != tk.a) out[k++] = tk.b;
    if (extra[t] >= 0 && extra[t] != tk.a && extra[t] != tk.b) out[k++] = extra[t];
    return k;
  };

  // 2. stages = (window, level), tasks in id order inside a stage
  std::vector<int32_t> order;
  order.reserve(T);
  for (int32_t t = 0; t < T; ++t)
    if (task_window[t] >= 0 && !skip[t]) order.push_back(t);
  std::stable_sort(order.begin(), order.end(), [&](int32_t x, int32_t y) {
    if (task_window[x] != task_window[y]) return task_window[x] < task_window[y];
    return plevel[x] < plevel[y];
  });
  std::vector<std::pair<int32_t, int32_t>> stages;  // [begin, end) in order
  for (size_t i = 0; i < order.size();) {
    size_t j = i;
    while (j < order.size() && task_window[order[j]] == task_window[order[i]] &&
           plevel[order[j]] == plevel[order[i]])
      ++j;
    stages.push_back({(int32_t)i, (int32_t)j});
    i = j;
  }

  PlanState S(ctx, in, plan);
  S.mask.assign(NT, 0);
  S.on_host.assign(NT, 0);
  S.uses_left.assign(NT, 0);
  S.use_stages.assign(NT, {});
  for (int32_t s = 0; s < (int32_t)stages.size(); ++s)
    for (int32_t i = stages[s].first; i < stages[s].second; ++i) {
      int32_t ops[3];
      const int k = operands(order[i], ops);
      for (int j = 0; j < k; ++j) {
        const int32_t op = ops[j];
        ++S.uses_left[op];
        if (S.use_stages[op].empty() || S.use_stages[op].back() != s) S.use_stages[op].push_back(s);
      }
    }
  S.res.assign(n, {});
  S.res_pos.assign(n, std::vector<int32_t>(NT, -1));
  S.pin.assign(n, std::vector<int32_t>(NT, -1));
  S.epoch.assign(n, 0);
  S.mem.assign(n, 0);
  S.st_flops.assign(n, 0);
  S.st_h2d.assign(n, 0);
  S.st_p2p.assign(n, 0);
  S.st_d2h.assign(n, 0);
  for (int g = 0; g < n && g < (int)in.initial_nodes.size(); ++g)
    for (int32_t x : in.initial_nodes[g])
      if (x >= 0 && x < NT && !((S.mask[x] >> g) & 1)) S.add_res(g, x);

  Scheduler sched(n, in.policy, in.reuse_bound, in.budget);
  const bool affinity = in.policy == MICCO_POLICY_MICCO_AFFINITY;  // last consumer's GPU first
  std::vector<int32_t> last_gpu(affinity ? NT : 0, -1);
  std::vector<std::vector<int32_t>> chunk(n);
  auto flush = [&](int g) {
    for (int32_t t : chunk[g]) S.emit(PlanOp::COMPUTE, g, -1, t);
    S.emit(PlanOp::FLUSH, g, -1, -1);
    chunk[g].clear();
    ++S.epoch[g];
  };

  // One stage (a vector of independent pairs): schedule, simulate the cache, emit the ops,
  // release dead operands.  Returns the stage's modelled time (max over GPUs).
  double stage_overlap_s = 0;  // the last run_stage's overlapped-copies model
  auto run_stage = [&](int32_t s) -> double {
    S.stage = s;
    sched.begin_vector(stages[s].second - stages[s].first);
    std::fill(S.st_flops.begin(), S.st_flops.end(), 0.0);
    std::fill(S.st_h2d.begin(), S.st_h2d.end(), 0.0);
    std::fill(S.st_p2p.begin(), S.st_p2p.end(), 0.0);
    std::fill(S.st_d2h.begin(), S.st_d2h.end(), 0.0);
    for (int32_t i = stages[s].first; i < stages[s].second; ++i) {
      const int32_t t = order[i];
      const TaskRec &tk = ctx.tasks[t];
      const int32_t a = tk.a, b = tk.b;
      const bool same = (b < 0 || b == a);
      const TensorRec &out = ctx.tensors[tk.out];
      const int32_t y = extra[t];  // fused dot partner (read in the epilogue), or -1
      const bool has_y = y >= 0 && y != a && y != b;
      SchedPair p;
      p.m1 = S.mask[a];
      p.m2 = same ? S.mask[a] : S.mask[b];
      p.same = same;
      p.b1 = S.bytes(a);
      p.b2 = same ? 0 : S.bytes(b);
      p.bout = (out.rank > 0 && y < 0) ? S.bytes(tk.out) : 0;
      p.flops = tk.flops + (y >= 0 ? ctx.tasks[plan.fused_dot[t]].flops : 0.0);
      if (has_y) { p.m3 = S.mask[y]; p.b3 = S.bytes(y); }
      if (affinity) p.pref = last_gpu[a] >= 0 ? last_gpu[a] : (same ? -1 : last_gpu[b]);
      sched.mem = S.mem;
      const int g = sched.decide(p);
      if (affinity) { last_gpu[a] = g; if (!same) last_gpu[b] = g; }
      const uint64_t bit = 1ULL << g;
      auto need_bytes = [&]() {
        int64_t need = p.bout;
        if (!(S.mask[a] & bit)) need += p.b1;
        if (!same && !(S.mask[b] & bit)) need += p.b2;
        if (has_y && !(S.mask[y] & bit)) need += S.bytes(y);
        return need;
      };
      // pin operands so the eviction below never drops them
      S.pin[g][a] = S.epoch[g];
      if (!same) S.pin[g][b] = S.epoch[g];
      if (has_y) S.pin[g][y] = S.epoch[g];
      if (!S.make_room(g, need_bytes())) {
        flush(g);  // split the stage: run what is pinned, then retry with this pair only
        S.pin[g][a] = S.epoch[g];
        if (!same) S.pin[g][b] = S.epoch[g];
        if (has_y) S.pin[g][y] = S.epoch[g];
        if (!S.make_room(g, need_bytes()))
          fail(MICCO_ERR_OOM, "planner: one contraction's operands and output (" +
                                  std::to_string(need_bytes()) + " B) exceed the GPU budget (" +
                                  std::to_string(in.budget[g]) + " B)");
      }
      if (S.mask[a] & bit) ++plan.cache_hits; else S.fetch(g, a);
      if (!same) { if (S.mask[b] & bit) ++plan.cache_hits; else S.fetch(g, b); }
      if (has_y) { if (S.mask[y] & bit) ++plan.cache_hits; else S.fetch(g, y); }
      if (out.rank > 0 && y < 0) {
        S.add_res(g, tk.out);
        S.pin[g][tk.out] = S.epoch[g];
      }
      sched.account(g, p);
      plan.task_gpu[t] = g;
      if (y >= 0) plan.task_gpu[plan.fused_dot[t]] = g;
      plan.gpu_flops[g] += p.flops;
      plan.flops += p.flops;
      S.st_flops[g] += p.flops;
      chunk[g].push_back(t);
    }
    for (int g = 0; g < n; ++g)
      if (!chunk[g].empty()) flush(g);
    // release operands whose last consumer ran
    for (int32_t i = stages[s].first; i < stages[s].second; ++i) {
      int32_t ops[3];
      const int k = operands(order[i], ops);
      for (int j = 0; j < k; ++j)
        if (--S.uses_left[ops[j]] == 0) S.release(ops[j]);
    }
    double worst = 0, worst_ov = 0;
    for (int g = 0; g < n; ++g) {
      const double tf = S.st_flops[g] / in.flops_per_s, th = (S.st_h2d[g] + S.st_d2h[g]) / (in.host_gbs * 1e9),
                   tp = S.st_p2p[g] / (in.peer_gbs * 1e9);
      worst = std::max(worst, tf + th + tp);
      // the executor's copy and peer streams overlap the kernels: the optimistic bound
      worst_ov = std::max(worst_ov, std::max(tf, std::max(th, tp)));
    }
    stage_overlap_s = worst_ov;
    return worst;
  };

  // Per-vector features (core.h kBoundFeatures), from the state before the stage runs.
  auto stage_features = [&](int32_t s, double *f) {
    int64_t slots = 0, repeated = 0, resident = 0;
    double bytes = 0;
    std::vector<int32_t> seen;
    for (int32_t i = stages[s].first; i < stages[s].second; ++i) {
      int32_t ops[3];
      const int k = operands(order[i], ops);
      for (int j = 0; j < k; ++j) seen.push_back(ops[j]);
    }
    std::vector<int32_t> sorted = seen;
    std::sort(sorted.begin(), sorted.end());
    for (int32_t x : seen) {
      ++slots;
      bytes += (double)S.bytes(x);
      auto r = std::equal_range(sorted.begin(), sorted.end(), x);
      if (r.second - r.first >= 2) ++repeated;
      if (S.mask[x]) ++resident;
    }
    const int64_t pairs = stages[s].second - stages[s].first;
    double pressure = 0;
    for (int g = 0; g < n; ++g) pressure = std::max(pressure, (double)S.mem[g] / (double)in.budget[g]);
    f[0] = (double)((pairs + n - 1) / n);
    f[1] = std::log2(std::max(1.0, bytes / std::max<int64_t>(1, slots)));
    f[2] = slots ? (double)repeated / (double)slots : 0.0;
    f[3] = slots ? (double)resident / (double)slots : 0.0;
    f[4] = (double)n;
    f[5] = pressure;
  };

  // Snapshot of everything a stage mutates, for the per-stage bound sweep.
  struct Snap {
    std::vector<uint64_t> mask;
    std::vector<char> on_host;
    std::vector<int32_t> uses_left, epoch;
    std::vector<std::vector<int32_t>> res, res_pos, pin;
    std::vector<int64_t> mem, peak;
    std::vector<double> gpu_flops;
    size_t n_ops;
    int64_t h2d, p2p, d2h, ev, hits;
    double flops;
  };
  auto save = [&](Snap &z) {
    z.mask = S.mask; z.on_host = S.on_host; z.uses_left = S.uses_left; z.epoch = S.epoch;
    z.res = S.res; z.res_pos = S.res_pos; z.pin = S.pin; z.mem = S.mem; z.peak = plan.gpu_peak_bytes;
    z.gpu_flops = plan.gpu_flops; z.n_ops = plan.ops.size();
    z.h2d = plan.bytes_h2d; z.p2p = plan.bytes_p2p; z.d2h = plan.bytes_d2h; z.ev = plan.evictions;
    z.hits = plan.cache_hits; z.flops = plan.flops;
  };
  auto restore = [&](const Snap &z) {
    S.mask = z.mask; S.on_host = z.on_host; S.uses_left = z.uses_left; S.epoch = z.epoch;
    S.res = z.res; S.res_pos = z.res_pos; S.pin = z.pin; S.mem = z.mem; plan.gpu_peak_bytes = z.peak;
    plan.gpu_flops = z.gpu_flops; plan.ops.resize(z.n_ops);
    plan.bytes_h2d = z.h2d; plan.bytes_p2p = z.p2p; plan.bytes_d2h = z.d2h; plan.evictions = z.ev;
    plan.cache_hits = z.hits; plan.flops = z.flops;
  };

  const bool per_stage = in.bound_mode != BOUNDS_FIXED && n > 1 &&
                         (in.policy == MICCO_POLICY_MICCO || in.policy == MICCO_POLICY_MICCO_AFFINITY);
  double predicted = 0, predicted_ov = 0;
  if (in.stream) in.stream->publish_fused(plan.fused_dot);
  for (int32_t s = 0; s < (int32_t)stages.size(); ++s) {
    double f[kBoundFeatures];
    stage_features(s, f);
    plan.stage_features.insert(plan.stage_features.end(), f, f + kBoundFeatures);
    int32_t bd[3] = {in.reuse_bound[0], in.reuse_bound[1], in.reuse_bound[2]};
    if (per_stage && in.bound_mode == BOUNDS_REGRESSION) {
      predict_bounds(f, bd);
    } else if (per_stage) {  // BOUNDS_STAGE_SWEEP: try {0,1,2}^3 on this stage, keep the cheapest
      Snap z;
      save(z);
      const Scheduler sched0 = sched;
      double best = 0;
      bool have = false;
      for (int c = 0; c < 27; ++c) {
        const int32_t cand[3] = {c / 9, (c / 3) % 3, c % 3};
        sched.set_bounds(cand);
        const double cost = run_stage(s);
        if (!have || cost < best * (1 - 1e-12)) { best = cost; have = true; for (int i = 0; i < 3; ++i) bd[i] = cand[i]; }
        restore(z);
        sched = sched0;
      }
    }
    sched.set_bounds(bd);
    plan.stage_bounds.insert(plan.stage_bounds.end(), bd, bd + 3);
    predicted += run_stage(s);
    predicted_ov += stage_overlap_s;
    if (in.stream) in.stream->publish_ops(plan.ops);  // this stage's ops are final
  }
  if (in.keep_inputs)
    for (int32_t x = 0; x < NT; ++x)
      if (S.mask[x] && ctx.tensors[x].node >= 0) plan.final_nodes.push_back({x, S.mask[x]});
  plan.n_stages = (int64_t)stages.size();
  plan.predicted_s = predicted;
  plan.predicted_overlap_s = predicted_ov;
  double mx = 0, sum = 0;
  for (double f : plan.gpu_flops) { mx = std::max(mx, f); sum += f; }
  plan.max_over_mean_load = sum > 0 ? mx / (sum / n) : 1.0;
  return plan;
}

int32_t choose_window(const Context &ctx, PlanInput in) {
  if (in.window_graphs > 0) return in.window_graphs;
  // A window's stages are level-synchronous, so all the intermediates of its first level are
  // live at once: under a tight budget a large window spills what a smaller one would not
  // (C5 at 25 GB: W = 256 moves 178 GB over PCIe per execute, W = 128 0.4 GB).  Take the
  // largest W in {256·n, 128·n, ..., 1} that a smaller W does not beat by more than 1% in the
  // cost model (which prices host bytes); stop at the first plan that spills nothing (a smaller
  // window only bounds the live set of intermediates).  Stages stay as large as the
  // budget allows (fewer, larger grouped launches).
  in.stream = nullptr;
  // The first candidate is 256 graphs per GPU: a stage then gives each GPU as many pairs as a
  // one-GPU stage (grouped launches of the same size; an 8-GPU weak-scaling plan has 81
  // instead of 628 stages).
  const int32_t w0 = 256 * std::max(1, in.n_gpus);
  int32_t best_w = w0;
  double best = 0;
  bool have = false;
  for (int32_t W = w0; W >= 1; W /= 2) {
    in.window_graphs = W;
    const Plan p = make_plan(ctx, in);
    if (!have || p.predicted_s < best * 0.99) {
      best = p.predicted_s;
      best_w = W;
      have = true;
    }
    if (p.bytes_d2h == 0) break;  // no spill (evicting dead or replicated tensors is cheap)
  }
  return best_w;
}

Plan make_plan_auto(const Context &ctx, PlanInput in) {
  if (in.n_gpus == 1 || in.policy == MICCO_POLICY_ROUND_ROBIN || in.policy == MICCO_POLICY_LEAST_LOADED ||
      in.policy == MICCO_POLICY_MICCO_NAIVE) {
    for (int i = 0; i < 3; ++i) in.reuse_bound[i] = 0;
    return make_plan(ctx, in);
  }
  // Sweep {0,1,2}^3 (a superset of the paper's 13 sets, L355) through
  // the planner's cost model and keep the cheapest plan (ties: lexicographically smallest).
  Plan best;
  bool have = false;
  for (int b0 = 0; b0 < 3; ++b0)
    for (int b1 = 0; b1 < 3; ++b1)
      for (int b2 = 0; b2 < 3; ++b2) {
        in.reuse_bound[0] = b0; in.reuse_bound[1] = b1; in.reuse_bound[2] = b2;
        Plan p = make_plan(ctx, in);
        if (!have || p.predicted_s < best.predicted_s * (1 - 1e-12)) { best = std::move(p); have = true; }
      }
  return best;
}

}  // namespace micco
