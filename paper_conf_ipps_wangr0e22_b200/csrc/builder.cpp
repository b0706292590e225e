// builder.cpp — graph validation, decomposition into pairwise hadron contractions, and
// hash-consing of shared contractions into one global task DAG.
//
// a graph is contracted by reducing "one edge after another";
// each reduction is a tensor contraction between hadron nodes.  L23: "repeated hadron nodes
// appear frequently because of overlapped reduction paths among multiple contraction graphs"
// — the same (operand, operand, contracted legs) step is interned once here, so a shared
// intermediate is computed once for every graph that needs it.
#include <algorithm>
#include <functional>
#include <numeric>
#include <string>

#include "core.h"
#include "layout.h"

namespace micco {

uint64_t content_hash(const double *data, int64_t n_doubles) {
  const uint64_t *w = reinterpret_cast<const uint64_t *>(data);
  uint64_t h0 = 0x243F6A8885A308D3ULL, h1 = 0x13198A2E03707344ULL;
  int64_t i = 0;
  for (; i + 1 < n_doubles; i += 2) {
    h0 = (h0 ^ w[i]) * 0x100000001B3ULL;
    h1 = (h1 ^ w[i + 1]) * 0x100000001B3ULL;
    h0 = (h0 << 29) | (h0 >> 35);
    h1 = (h1 << 31) | (h1 >> 33);
  }
  if (i < n_doubles) h0 = (h0 ^ w[i]) * 0x100000001B3ULL;
  uint64_t h = h0 ^ (h1 * 0x9E3779B97F4A7C15ULL) ^ (uint64_t)n_doubles;
  h ^= h >> 33; h *= 0xFF51AFD7ED558CCDULL; h ^= h >> 33;
  return h;
}

int32_t add_node_tensor(Context &ctx, int32_t node) {
  const NodeRec &n = ctx.nodes[node];
  TensorRec t;
  t.rank = n.rank;
  for (int i = 0; i < n.rank; ++i) t.dim[i] = n.N;
  t.slice_elems = n.slice_elems;
  t.node = node;
  t.level = 0;
  ctx.tensors.push_back(t);
  return (int32_t)ctx.tensors.size() - 1;
}

namespace {

struct Comp {
  int32_t tensor;                 // committed tensor id, or -1 while dry-running
  int32_t rank;
  int32_t leg[2 * kMaxRank + 4];  // global leg id = inst * 8 + position
  int32_t dim[2 * kMaxRank + 4];
  int32_t level;
  bool alive;
  double flops;                   // no-dedup flops of the steps merged into this component
};

struct Step {  // one pairwise reduction chosen for a graph
  int32_t ca, cb;   // component indices (cb = -1: trace)
  int8_t c;
  int8_t pa[kMaxRank], pb[kMaxRank];
};

int64_t prod(const int32_t *d, int n) {
  int64_t s = 1;
  for (int i = 0; i < n; ++i) s *= d[i];
  return s;
}

int find_leg(const Comp &c, int32_t gleg) {
  for (int i = 0; i < c.rank; ++i)
    if (c.leg[i] == gleg) return i;
  return -1;
}

}  // namespace

void build_graph(Context &ctx, int32_t n_inst, const int64_t *node_ids, int32_t n_edges,
                 const micco_edge *edges, const int32_t *order, double cre, double cim) {
  if (n_inst < 1 || !node_ids) fail(MICCO_ERR_ARG, "add_graph: need n_inst >= 1 and node_ids");
  if (n_edges < 0 || (n_edges > 0 && !edges)) fail(MICCO_ERR_ARG, "add_graph: bad edges");
  if (n_inst > 1 << 20) fail(MICCO_ERR_ARG, "add_graph: too many instances");
  std::vector<int32_t> rank(n_inst), N(n_inst);
  int64_t legs_total = 0;
  for (int u = 0; u < n_inst; ++u) {
    if (node_ids[u] < 0 || node_ids[u] >= (int64_t)ctx.nodes.size())
      fail(MICCO_ERR_ARG, "add_graph: node id " + std::to_string(node_ids[u]) + " does not exist");
    rank[u] = ctx.nodes[node_ids[u]].rank;
    N[u] = ctx.nodes[node_ids[u]].N;
    legs_total += rank[u];
  }
  if (legs_total != 2 * (int64_t)n_edges)
    fail(MICCO_ERR_GRAPH, "add_graph: the edges must match every leg exactly once (" +
                              std::to_string(legs_total) + " legs, " + std::to_string(n_edges) + " edges)");
  std::vector<int32_t> seen((size_t)n_inst * 8, 0);
  for (int e = 0; e < n_edges; ++e) {
    const micco_edge &E = edges[e];
    if (E.u < 0 || E.u >= n_inst || E.v < 0 || E.v >= n_inst)
      fail(MICCO_ERR_GRAPH, "add_graph: edge " + std::to_string(e) + " names a missing instance");
    if (E.p < 0 || E.p >= rank[E.u] || E.q < 0 || E.q >= rank[E.v])
      fail(MICCO_ERR_GRAPH, "add_graph: edge " + std::to_string(e) + " leg index >= rank");
    if (E.u == E.v && E.p == E.q) fail(MICCO_ERR_GRAPH, "add_graph: edge joins a leg to itself");
    if (seen[E.u * 8 + E.p]++ || seen[E.v * 8 + E.q]++)
      fail(MICCO_ERR_GRAPH, "add_graph: a leg is matched twice (edge " + std::to_string(e) + ")");
    if (N[E.u] != N[E.v]) fail(MICCO_ERR_GRAPH, "add_graph: joined legs have unequal N");
    if (E.u == E.v && rank[E.u] != 2)
      fail(MICCO_ERR_UNSUPPORTED, "add_graph: baryon partial traces are not supported");
  }
  if (order) {
    std::vector<char> hit(n_edges, 0);
    for (int i = 0; i < n_edges; ++i) {
      if (order[i] < 0 || order[i] >= n_edges || hit[order[i]])
        fail(MICCO_ERR_GRAPH, "add_graph: order is not a permutation of the edges");
      hit[order[i]] = 1;
    }
  }

  // Canonical sub-network hashing: a connected component whose hadron
  // nodes and wiring equal, up to relabeling its instances, a component interned by an earlier
  // graph has the same value (overlapped reduction paths), whatever tree either
  // was contracted by — e.g. tr(ABC) and tr(BCA).  When every component of this graph is such a
  // repeat, the graph reuses the earlier scalars and no task is built; otherwise the graph is
  // decomposed as usual and its components are recorded.  The key: instances sorted by node id
  // (ties: every order within a group of equal nodes), then the sorted normalised edge list;
  // the smallest over the tie orders.  Components with more than 5040 tie orders keep no key.
  std::vector<int32_t> comp_root(n_inst);
  {
    std::vector<int32_t> parent(n_inst);
    std::iota(parent.begin(), parent.end(), 0);
    auto find = [&](int32_t x) {  // iterative, path halving (graphs may have 2^20 instances)
      while (parent[x] != x) x = parent[x] = parent[parent[x]];
      return x;
    };
    for (int e = 0; e < n_edges; ++e) parent[find(edges[e].u)] = find(edges[e].v);
    for (int u = 0; u < n_inst; ++u) comp_root[u] = find(u);
  }
  // members and edges of each component, bucketed once
  std::vector<std::vector<int32_t>> comp_members(n_inst), comp_edges(n_inst);
  for (int u = 0; u < n_inst; ++u) comp_members[comp_root[u]].push_back(u);
  for (int e = 0; e < n_edges; ++e) comp_edges[comp_root[edges[e].u]].push_back(e);
  std::vector<int32_t> pos(n_inst, -1);
  auto component_key = [&](int32_t root) -> std::string {
    std::vector<int32_t> mem = comp_members[root];
    std::stable_sort(mem.begin(), mem.end(), [&](int32_t x, int32_t y) { return node_ids[x] < node_ids[y]; });
    // tie groups (equal node ids) are permuted among themselves
    std::vector<std::pair<int, int>> groups;
    double orders = 1;
    for (size_t i = 0; i < mem.size();) {
      size_t j = i;
      while (j < mem.size() && node_ids[mem[j]] == node_ids[mem[i]]) ++j;
      groups.push_back({(int)i, (int)j});
      for (size_t k = 2; k <= j - i; ++k) orders *= (double)k;
      i = j;
    }
    if (orders > 5040) return std::string();
    std::vector<int64_t> best;
    std::vector<int32_t> cur = mem;
    std::vector<std::pair<int64_t, int64_t>> ek;
    std::function<void(size_t)> rec = [&](size_t gi) {
      if (gi == groups.size()) {
        for (size_t i = 0; i < cur.size(); ++i) pos[cur[i]] = (int32_t)i;
        std::vector<int64_t> key;
        key.push_back((int64_t)cur.size());
        for (int32_t u : cur) key.push_back(node_ids[u]);
        ek.clear();
        for (int32_t e : comp_edges[root]) {
          const micco_edge &E = edges[e];
          int64_t a = (int64_t)pos[E.u] * 8 + E.p, b = (int64_t)pos[E.v] * 8 + E.q;
          if (a > b) std::swap(a, b);
          ek.push_back({a, b});
        }
        std::sort(ek.begin(), ek.end());
        for (const auto &ab : ek) { key.push_back(ab.first); key.push_back(ab.second); }
        if (best.empty() || key < best) best.swap(key);
        return;
      }
      auto [b, e] = groups[gi];
      std::sort(cur.begin() + b, cur.begin() + e);
      do rec(gi + 1);
      while (std::next_permutation(cur.begin() + b, cur.begin() + e));
    };
    rec(0);
    return std::string(reinterpret_cast<const char *>(best.data()), best.size() * sizeof(int64_t));
  };
  std::vector<int32_t> roots;
  for (int u = 0; u < n_inst; ++u)
    if (comp_root[u] == u) roots.push_back(u);
  std::vector<std::string> keys(roots.size());
  std::vector<int32_t> key_of_root(n_inst, -1);
  for (size_t i = 0; i < roots.size(); ++i) key_of_root[roots[i]] = (int32_t)i;
  {
    bool all_known = true;
    for (size_t i = 0; i < roots.size(); ++i) {
      keys[i] = component_key(roots[i]);
      if (keys[i].empty() || !ctx.component_by_key.count(keys[i])) all_known = false;
    }
    if (all_known) {
      GraphRec g;
      g.coef_re = cre;
      g.coef_im = cim;
      g.comp_begin = (int32_t)ctx.graph_scalars.size();
      double fl = 0;
      for (const std::string &k : keys) {
        const auto &hit = ctx.component_by_key.at(k);
        ctx.graph_scalars.push_back(hit.first);
        fl += hit.second;
      }
      g.comp_end = (int32_t)ctx.graph_scalars.size();
      g.flops_no_dedup = fl;
      ctx.graphs.push_back(g);
      ctx.component_dedup_hits += (int64_t)keys.size();
      return;
    }
  }

  // Two passes over the same decomposition: a dry run that picks the steps and validates
  // ranks and layouts (so a failing graph leaves the DAG untouched), then the commit that
  // replays the dry run's steps and interns tasks.  The dry run predicts the ids the commit
  // will give new tensors (they are appended in step order), so hash-consing keys — and the
  // reuse-aware order, which looks them up — are identical in both passes.
  const bool reorder = ctx.opt.reorder != 0;
  std::vector<int32_t> chosen;  // edge picked at each step by the dry run
  chosen.reserve(n_edges);
  for (int pass = 0; pass < 2; ++pass) {
    const bool commit = pass == 1;
    std::vector<Comp> comps(n_inst);
    std::vector<int32_t> comp_of(n_inst), n_members(n_inst, 1);
    for (int u = 0; u < n_inst; ++u) {
      Comp &c = comps[u];
      c.tensor = ctx.nodes[node_ids[u]].tensor;
      c.rank = rank[u];
      for (int p = 0; p < rank[u]; ++p) { c.leg[p] = u * 8 + p; c.dim[p] = N[u]; }
      c.level = 0;
      c.alive = true;
      c.flops = 0;
      comp_of[u] = u;
    }
    std::vector<char> done(n_edges, 0);
    double flops_nd = 0;
    int steps_left = n_edges;
    int32_t next_new = (int32_t)ctx.tensors.size();  // dry run: id the commit will assign
    std::unordered_map<TaskKey, int32_t, TaskKeyHash> fresh;  // dry run: keys new in this graph

    auto plan_step = [&](int e, Step &st, int &res_rank, int64_t &res_size, int64_t &kdim) {
      const micco_edge &E = edges[e];
      int a = comp_of[E.u], b = comp_of[E.v];
      st.c = 0;
      if (a == b) {  // meson self-edge: full trace (validated above)
        st.ca = a; st.cb = -1; st.c = 1;
        st.pa[0] = (int8_t)find_leg(comps[a], E.u * 8 + E.p);
        st.pb[0] = (int8_t)find_leg(comps[a], E.v * 8 + E.q);
        res_rank = comps[a].rank - 2;
        res_size = 1;
        kdim = comps[a].dim[st.pa[0]];
        return;
      }
      st.ca = a; st.cb = b;
      int8_t pa[16], pb[16];
      int c = 0;
      for (int f = 0; f < n_edges; ++f) {
        if (done[f]) continue;
        const micco_edge &F = edges[f];
        int cu = comp_of[F.u], cv = comp_of[F.v];
        if (cu == a && cv == b) {
          pa[c] = (int8_t)find_leg(comps[a], F.u * 8 + F.p); pb[c] = (int8_t)find_leg(comps[b], F.v * 8 + F.q);
        } else if (cu == b && cv == a) {
          pa[c] = (int8_t)find_leg(comps[a], F.v * 8 + F.q); pb[c] = (int8_t)find_leg(comps[b], F.u * 8 + F.p);
        } else {
          continue;
        }
        if (++c > kMaxRank) break;
      }
      res_rank = comps[a].rank + comps[b].rank - 2 * c;
      if (c > kMaxRank) { res_rank = 99; return; }
      // sort pairs by position in a (canonical key)
      int idx[kMaxRank];
      std::iota(idx, idx + c, 0);
      std::sort(idx, idx + c, [&](int x, int y) { return pa[x] < pa[y]; });
      kdim = 1;
      for (int i = 0; i < c; ++i) { st.pa[i] = pa[idx[i]]; st.pb[i] = pb[idx[i]]; kdim *= comps[a].dim[st.pa[i]]; }
      for (int i = c; i < kMaxRank; ++i) { st.pa[i] = 0; st.pb[i] = 0; }
      st.c = (int8_t)c;
      res_size = prod(comps[a].dim, comps[a].rank) * prod(comps[b].dim, comps[b].rank) / (kdim * kdim);
    };
    // Canonical operand order for hash-consing: the lower tensor id is the left operand
    // (a contraction and its mirror image are one task; the component keeps track of
    // which legs the result carries, so the graph value is unchanged).
    auto canonical = [&](Step &st) {
      if (st.cb < 0 || comps[st.cb].tensor >= comps[st.ca].tensor) return;
      std::swap(st.ca, st.cb);
      int8_t pa2[kMaxRank], pb2[kMaxRank];
      int idx[kMaxRank];
      std::iota(idx, idx + st.c, 0);
      std::sort(idx, idx + st.c, [&](int x, int y) { return st.pb[x] < st.pb[y]; });
      for (int i = 0; i < st.c; ++i) { pa2[i] = st.pb[idx[i]]; pb2[i] = st.pa[idx[i]]; }
      for (int i = 0; i < st.c; ++i) { st.pa[i] = pa2[i]; st.pb[i] = pb2[i]; }
    };
    auto make_key = [&](const Step &st) {
      TaskKey key{};
      key.a = comps[st.ca].tensor;
      key.b = st.cb < 0 ? -1 : comps[st.cb].tensor;
      key.c = st.c;
      std::memcpy(key.pa, st.pa, kMaxRank);
      std::memcpy(key.pb, st.pb, kMaxRank);
      return key;
    };
    auto interned = [&](const TaskKey &key) {
      return ctx.task_by_key.count(key) > 0 || (!commit && fresh.count(key) > 0);
    };

    for (int step = 0; steps_left > 0; ++step) {
      int e = -1;
      Step st{};
      int rr = 0;
      int64_t rs = 0, kd = 0;
      if (commit) {  // replay the dry run's choice
        e = chosen[step];
        plan_step(e, st, rr, rs, kd);
      } else if (order && !reorder) {
        if (step >= n_edges) break;
        e = order[step];
        if (done[e]) continue;
        plan_step(e, st, rr, rs, kd);
      } else {
        // greedy (order NULL): smallest result, then fewest flops, then lowest edge index.
        // reuse-aware (options.reorder): an already-interned step first
        // (free: dedup hit), then the same size/flops rule, then the fewest hadron nodes in
        // the result — node-pair products are shared by the most graphs.
        int64_t best_s = 0;
        double best_f = 0;
        int best_hit = 0, best_m = 0;
        for (int f = 0; f < n_edges; ++f) {
          if (done[f]) continue;
          Step s2{};
          int r2;
          int64_t sz, k2;
          plan_step(f, s2, r2, sz, k2);
          if (r2 > kMaxRank) continue;
          double fl = (double)sz * (double)k2;
          int hit = 0, m = 0;
          if (reorder) {
            Step s3 = s2;
            canonical(s3);
            hit = interned(make_key(s3)) ? 0 : 1;
            m = n_members[s2.ca] + (s2.cb >= 0 ? n_members[s2.cb] : 0);
          }
          bool better = e < 0 || hit < best_hit ||
                        (hit == best_hit && (sz < best_s || (sz == best_s && (fl < best_f || (fl == best_f && m < best_m)))));
          if (better) {
            e = f; st = s2; rr = r2; rs = sz; kd = k2; best_s = sz; best_f = fl; best_hit = hit; best_m = m;
          }
        }
        if (e < 0) { plan_step(0, st, rr, rs, kd); rr = 99; }
      }
      if (rr > kMaxRank)
        fail(MICCO_ERR_UNSUPPORTED, "add_graph: the reduction order creates an intermediate of rank > 4");
      if (st.cb >= 0) {  // the kernels must be able to read both operands in place
        const Comp &A = comps[st.ca], &B = comps[st.cb];
        bool ok;
        const long long lim = (1LL << 31) - 1;  // the kernels keep per-slice offsets in 32 bits
        bool fits = true;
        if (rr > 0) {
          GemmLayout gl;
          ok = gemm_layout(A.rank, A.dim, B.rank, B.dim, st.c, st.pa, st.pb, gl);
          // (the executor's limits, checked here so a graph the kernels cannot run is refused
          // at add_graph, not part-way through an execute; 64 × 32 is the smallest tile)
          if (ok)
            fits = gl.sliceA <= lim && gl.sliceB <= lim && gl.sliceC <= lim &&
                   (long long)ctx.Lt * gl.Mo * gl.No * ((gl.Mi + 63) / 64) * ((gl.Ni + 31) / 32) < (1LL << 32);
        } else {
          DotLayout dl;
          ok = dot_layout(A.rank, A.dim, B.rank, B.dim, st.c, st.pa, st.pb, dl);
          if (ok) fits = dl.sliceA <= lim && dl.sliceB <= lim;
        }
        if (!ok) fail(MICCO_ERR_UNSUPPORTED, "add_graph: contraction layout not supported by the kernels");
        if (!fits) fail(MICCO_ERR_UNSUPPORTED, "add_graph: a tensor slice exceeds 2^31 elements (kernel limit)");
      }
      if (!commit) chosen.push_back(e);
      // mark contracted edges done
      {
        const micco_edge &E = edges[e];
        int a = comp_of[E.u], b = comp_of[E.v];
        for (int f = 0; f < n_edges; ++f) {
          if (done[f]) continue;
          const micco_edge &F = edges[f];
          int cu = comp_of[F.u], cv = comp_of[F.v];
          bool hit = (a == b) ? (f == e) : ((cu == a && cv == b) || (cu == b && cv == a));
          if (hit) { done[f] = 1; --steps_left; }
        }
      }
      canonical(st);
      Comp &A = comps[st.ca];
      Comp res{};
      res.alive = true;
      res.flops = A.flops + (st.cb >= 0 ? comps[st.cb].flops : 0.0);
      double step_flops;
      if (st.cb < 0) {  // trace
        res.rank = 0;
        res.level = A.level + 1;
        step_flops = 2.0 * (double)kd * ctx.Lt;
      } else {
        Comp &B = comps[st.cb];
        int r = 0;
        for (int i = 0; i < A.rank; ++i) {
          bool used = false;
          for (int j = 0; j < st.c; ++j) used |= st.pa[j] == i;
          if (!used) { res.leg[r] = A.leg[i]; res.dim[r] = A.dim[i]; ++r; }
        }
        for (int i = 0; i < B.rank; ++i) {
          bool used = false;
          for (int j = 0; j < st.c; ++j) used |= st.pb[j] == i;
          if (!used) { res.leg[r] = B.leg[i]; res.dim[r] = B.dim[i]; ++r; }
        }
        res.rank = r;
        res.level = std::max(A.level, B.level) + 1;
        step_flops = 8.0 * (double)rs * (double)kd * ctx.Lt;
      }
      flops_nd += step_flops;
      res.flops += step_flops;
      res.tensor = -1;
      const TaskKey key = make_key(st);
      if (!commit) {  // predict the id the commit gives this step's result
        auto it = ctx.task_by_key.find(key);
        if (it != ctx.task_by_key.end()) {
          res.tensor = ctx.tasks[it->second].out;
        } else {
          auto jt = fresh.find(key);
          if (jt != fresh.end()) res.tensor = jt->second;
          else fresh.emplace(key, res.tensor = next_new++);
        }
      } else {
        auto it = ctx.task_by_key.find(key);
        if (it != ctx.task_by_key.end()) {
          res.tensor = ctx.tasks[it->second].out;
          ++ctx.dedup_hits;
        } else {
          TaskRec T;
          T.kind = st.cb < 0 ? TASK_TRACE : (res.rank == 0 ? TASK_DOT : TASK_GEMM);
          T.a = key.a;
          T.b = key.b;
          T.c = st.c;
          std::memcpy(T.pa, st.pa, kMaxRank);
          std::memcpy(T.pb, st.pb, kMaxRank);
          T.flops = step_flops;
          TensorRec out;
          out.rank = res.rank;
          for (int i = 0; i < res.rank; ++i) out.dim[i] = res.dim[i];
          out.slice_elems = prod(res.dim, res.rank);
          T.level = std::max(ctx.tensors[key.a].level, key.b >= 0 ? ctx.tensors[key.b].level : 0) + 1;
          out.level = T.level;
          out.task = (int32_t)ctx.tasks.size();
          if (out.rank == 0) out.scalar_slot = ctx.n_scalar_slots++;
          ctx.tensors.push_back(out);
          T.out = (int32_t)ctx.tensors.size() - 1;
          ctx.tasks.push_back(T);
          ctx.task_by_key.emplace(key, (int32_t)ctx.tasks.size() - 1);
          res.tensor = T.out;
        }
      }
      // merge: result replaces component ca; cb dies
      int ca = st.ca, cb = st.cb;
      comps[ca] = res;
      if (cb >= 0) {
        n_members[ca] += n_members[cb];
        comps[cb].alive = false;
        for (int u = 0; u < n_inst; ++u)
          if (comp_of[u] == cb) comp_of[u] = ca;
      }
    }
    for (int u = 0; u < n_inst; ++u)
      if (comps[u].alive && comps[u].rank != 0)
        fail(MICCO_ERR_GRAPH, "add_graph: graph did not contract to scalars");
    if (commit) {
      GraphRec g;
      g.coef_re = cre;
      g.coef_im = cim;
      g.comp_begin = (int32_t)ctx.graph_scalars.size();
      for (int u = 0; u < n_inst; ++u)
        if (comps[u].alive) {
          ctx.graph_scalars.push_back(comps[u].tensor);
          // record the component for canonical reuse (its members share comp_root)
          const std::string &k = keys[key_of_root[comp_root[u]]];
          if (!k.empty()) ctx.component_by_key.emplace(k, std::make_pair(comps[u].tensor, comps[u].flops));
        }
      g.comp_end = (int32_t)ctx.graph_scalars.size();
      g.flops_no_dedup = flops_nd;
      ctx.graphs.push_back(g);
    }
  }
}

}  // namespace micco
