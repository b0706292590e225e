"""Host-side tests of libmicco.so that need no GPU: the library loads and exports
every symbol include/micco.h declares; the builder's validation, dedup and
hash-consing; the planner's invariants; and the native scheduler against the
oracle (oracle/sched.py) decision for decision."""
import re
from pathlib import Path

import numpy as np
import pytest

import paper_conf_ipps_wangr0e22_b200 as M
from micco_inputs import workloads
from micco_inputs.gen import GraphSpec, NodeSpec, Workload
from oracle.sched import MiccoSchedulerOracle, Pair

ROOT = Path(__file__).resolve().parent.parent


@pytest.fixture(scope="module", autouse=True)
def _built():
    import sys
    sys.path.insert(0, str(ROOT / "tools"))
    from build import build_lib
    build_lib()


def test_exports_every_declared_symbol():
    hdr = (ROOT / "include" / "micco.h").read_text()
    declared = set(re.findall(r"MICCO_API\s+[\w\s\*]+?\b(micco_\w+)\s*\(", hdr))
    assert declared == set(M.EXPORTS), declared ^ set(M.EXPORTS)
    L = M.lib()
    for name in declared:
        assert hasattr(L, name), name


def _ctx(**kw):
    kw.setdefault("mem_budget_bytes", 1 << 30)
    return M.Context(**kw)


def test_node_dedup_by_content_and_lt_check():
    ctx = _ctx()
    a = np.arange(2 * 4 * 4, dtype=np.float64).reshape(2, 4, 4) + 1j
    i0 = ctx.add_node(a)
    i1 = ctx.add_node(a.copy())
    i2 = ctx.add_node(a + 1)
    assert i0 == i1 and i2 != i0
    with pytest.raises(M.MiccoError) as e:
        ctx.add_node(np.zeros((3, 4, 4), dtype=complex))
    assert e.value.status == -1  # Lt mismatch


def test_graph_validation_errors():
    ctx = _ctx()
    m = ctx.add_node(np.ones((1, 2, 2), dtype=complex))
    b = ctx.add_node(np.ones((1, 2, 2, 2), dtype=complex))
    cases = [
        ([m, m], [(0, 1, 1, 0)], None, -3),                      # unmatched legs
        ([m, m], [(0, 1, 1, 0), (0, 1, 1, 1)], None, -3),        # leg matched twice
        ([m, m], [(0, 2, 1, 0), (1, 1, 0, 0)], None, -3),        # leg index >= rank
        ([m, m], [(0, 1, 1, 0), (1, 1, 0, 0)], [0, 0], -3),      # order not a permutation
        ([b], [(0, 0, 0, 1)], None, -3),                          # odd legs
        ([b, m], [(0, 0, 0, 1), (0, 2, 1, 0), (1, 1, 1, 0)], None, -3),
    ]
    for inst, edges, order, code in cases:
        with pytest.raises(M.MiccoError) as e:
            ctx.add_graph(inst, edges, order)
        assert e.value.status == code, (edges, e.value)
    # baryon partial trace is unsupported
    with pytest.raises(M.MiccoError) as e:
        ctx.add_graph([b, m, b], [(0, 0, 0, 1), (0, 2, 1, 0), (1, 1, 2, 0), (2, 1, 2, 2)])
    assert e.value.status in (-3, -4)
    # a failing graph leaves no tasks behind
    st, _ = ctx.plan(1, [0, 0, 0]) if ctx.n_graphs else ({"unique_tasks": 0}, None)


def test_unequal_N_rejected():
    ctx = _ctx()
    a = ctx.add_node(np.ones((1, 2, 2), dtype=complex))
    b = ctx.add_node(np.ones((1, 3, 3), dtype=complex))
    with pytest.raises(M.MiccoError) as e:
        ctx.add_graph([a, b], [(0, 1, 1, 0), (1, 1, 0, 0)])
    assert e.value.status == -3


def test_hash_consing_counts():
    """tr(AB), tr(ABC), tr(ABD): the product A·B is one task shared by the last two
    (overlapping reduction paths), and tr(AB) is a dot."""
    ctx = _ctx()
    rng = np.random.default_rng(0)
    ids = [ctx.add_node(rng.standard_normal((1, 4, 4)) + 0j) for _ in range(4)]
    A, B, C, D = ids
    ctx.add_graph([A, B], workloads.meson_cycle_edges(2), [0, 1])
    ctx.add_graph([A, B, C], workloads.meson_cycle_edges(3), [0, 1, 2])
    ctx.add_graph([A, B, D], workloads.meson_cycle_edges(3), [0, 1, 2])
    st, _ = ctx.plan(1, [0, 0, 0])
    # tasks: dot(A,B), gemm(A,B), dot(AB,C), dot(AB,D)
    assert st["unique_tasks"] == 4 and st["n_gemm"] == 1 and st["n_dot"] == 3
    assert st["dedup_hits"] == 1
    # identical graph again: its one component is reused whole (canonical sub-network hashing)
    ctx.add_graph([A, B, C], workloads.meson_cycle_edges(3), [0, 1, 2])
    st2, _ = ctx.plan(1, [0, 0, 0])
    assert st2["unique_tasks"] == 4 and st2["component_dedup_hits"] == 1 and st2["dedup_hits"] == 1


def test_flops_accounting():
    """N×N×N complex GEMM = 8N³ flops per slice."""
    N, Lt = 8, 3
    ctx = _ctx()
    rng = np.random.default_rng(1)
    ids = [ctx.add_node(rng.standard_normal((Lt, N, N)) + 0j) for _ in range(3)]
    ctx.add_graph(ids, workloads.meson_cycle_edges(3), [0, 1, 2])
    st, _ = ctx.plan(1, [0, 0, 0])
    assert st["flops"] == 8 * N ** 3 * Lt + 8 * N * N * Lt
    assert st["flops_no_dedup"] == st["flops"]


def test_plan_stage_structure_and_invariants():
    wl = workloads.c2_meson_set(n_graphs=300, N=8, Lt=2, rate=0.5)
    ctx = _ctx(window_graphs=50)
    M.load_workload(ctx, wl)
    for n in (1, 2, 4, 8):
        st, assign = ctx.plan(n, [1, 1, 1], n_tasks=None)
        assert st["n_gpus"] == n
        st, assign = M.micco_plan(ctx.h, n, [1, 1, 1], n_tasks=st["unique_tasks"])
        assert np.all((assign >= 0) & (assign < n))  # every task assigned exactly once
        if n == 1:
            assert st["bytes_p2p"] == 0 and st["max_over_mean_load"] == 1.0
    # 6 windows × up to 3 levels
    assert st["n_stages"] <= 6 * 3


def test_tight_budget_forces_evictions_and_spills():
    wl = workloads.c2_meson_set(n_graphs=200, N=16, Lt=4, rate=0.7)
    node_bytes = 16 * 16 * 4 * 16
    big = _ctx(mem_budget_bytes=1 << 30, window_graphs=200)
    M.load_workload(big, wl)
    s_big, _ = big.plan(1, [0, 0, 0])
    small = _ctx(mem_budget_bytes=12 * node_bytes, window_graphs=200)
    M.load_workload(small, wl)
    s_small, _ = small.plan(1, [0, 0, 0])
    assert s_big["evictions"] == 0
    assert s_small["evictions"] > 0
    assert s_small["bytes_h2d"] > s_big["bytes_h2d"]
    # a budget below one task's working set is an OOM error
    tiny = _ctx(mem_budget_bytes=2 * node_bytes)
    M.load_workload(tiny, wl)
    with pytest.raises(M.MiccoError) as e:
        tiny.plan(1, [0, 0, 0])
    assert e.value.status == -5


def test_reuse_beats_round_robin_on_repetition_heavy_set():
    """On a repetition-heavy set MICCO moves fewer bytes than round-robin
    (BASELINE.json north_star; Fig. 2 L90)."""
    wl = workloads.c2_meson_set(n_graphs=600, N=16, Lt=4, rate=0.9, dist="gaussian")
    res = {}
    for pol in ("micco", "round_robin", "least_loaded", "micco_naive"):
        ctx = _ctx(policy=pol, window_graphs=64)
        M.load_workload(ctx, wl)
        st, _ = ctx.plan(4, [1, 2, 0] if pol == "micco" else None)
        res[pol] = st["bytes_h2d"] + st["bytes_p2p"]
    assert res["micco"] < res["round_robin"]
    assert res["micco"] <= res["micco_naive"]


def test_auto_bounds_sweep_picks_a_valid_set():
    wl = workloads.c2_meson_set(n_graphs=200, N=8, Lt=2, rate=0.8)
    ctx = _ctx(window_graphs=32)
    M.load_workload(ctx, wl)
    st, _ = ctx.plan(4, None)
    assert all(0 <= b <= 2 for b in st["reuse_bound"])


# ---------------------------------------------------------------- scheduler parity with the oracle


def _random_stream(rng, n_gpus, n_vec=6, n_tensors=40):
    vecs, nxt = [], 10_000
    for _ in range(n_vec):
        v = []
        for _ in range(int(rng.integers(1, 30))):
            t1, t2 = int(rng.integers(0, n_tensors)), int(rng.integers(0, n_tensors))
            fl = float(rng.integers(1, 5)) * 1e6
            v.append((t1, t2, nxt, fl, int(rng.integers(1, 4)) * 100, int(rng.integers(1, 4)) * 100, 100))
            nxt += 1
        vecs.append(v)
    res = [(int(rng.integers(0, n_tensors)), int(rng.integers(0, n_gpus))) for _ in range(int(rng.integers(0, 20)))]
    return vecs, res


@pytest.mark.parametrize("seed", range(30))
def test_native_scheduler_matches_oracle(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 9))
    bd = [int(x) for x in rng.integers(0, 3, size=3)]
    budget = float(rng.choice([1e30, 3000.0, 8000.0]))
    vecs, res = _random_stream(rng, n)
    O = MiccoSchedulerOracle(n, bd, budget)
    for t, g in res:
        if g not in O.res.setdefault(t, set()):
            O.res[t].add(g)
    got_o = O.run([[Pair(*p) for p in v] for v in vecs])
    got_n = M.micco_debug_schedule(n, bd, budget, vecs, resident=res)
    assert got_n == got_o


def test_reorder_reuse_aware_dedup():
    """options.reorder: on the C3 wiring the node-pair products
    S·R come first and are shared by many graphs, so the unique GEMMs drop > 2x (3.5x at 10k graphs) against
    the chain order; on C4 the chain order collapses to the greedy (c = 2 first) DAG; the
    graph count and the flops of the as-given DAG are unchanged by construction."""
    wl = workloads.c3_multi_meson(n_graphs=2000, N=4, Lt=1)
    counts = {}
    for reorder in (False, True):
        ctx = _ctx(reorder=reorder)
        M.load_workload(ctx, wl)
        st, _ = ctx.plan(1, [0, 0, 0])
        counts[reorder] = st
        ctx.close()
    assert counts[True]["n_gemm"] * 2 < counts[False]["n_gemm"], (counts[True]["n_gemm"], counts[False]["n_gemm"])
    assert counts[True]["flops"] < counts[False]["flops"]
    assert counts[True]["flops_no_dedup"] > 0
    c4 = {}
    for order, reorder in (("greedy", False), ("chain", False), ("chain", True)):
        ctx = _ctx(reorder=reorder)
        M.load_workload(ctx, workloads.c4_two_baryon(n_combos=4, N=3, Lt=1, order=order))
        c4[(order, reorder)] = ctx.plan(1, [0, 0, 0])[0]
        ctx.close()
    assert c4[("chain", True)]["n_gemm"] == c4[("greedy", False)]["n_gemm"] < c4[("chain", False)]["n_gemm"]


def test_reorder_dry_run_leaves_dag_untouched_on_failure():
    """The dry pass predicts tensor ids exactly; a graph that fails validation under
    reorder leaves no task behind."""
    ctx = _ctx(reorder=True)
    rng = np.random.default_rng(3)
    ids = [ctx.add_node(rng.standard_normal((1, 4, 4)) + 0j) for _ in range(3)]
    ctx.add_graph(ids, workloads.meson_cycle_edges(3), None)
    st0, _ = ctx.plan(1, [0, 0, 0])
    with pytest.raises(M.MiccoError):
        ctx.add_graph(ids, [(0, 1, 1, 0), (1, 1, 2, 0), (2, 1, 2, 0)], None)  # leg (2, 0) twice
    st1, _ = ctx.plan(1, [0, 0, 0])
    assert st1["unique_tasks"] == st0["unique_tasks"]
    ctx.add_graph([ids[1], ids[2], ids[0]], workloads.meson_cycle_edges(3), None)  # rotation: reused whole
    st2, _ = ctx.plan(1, [0, 0, 0])
    assert st2["unique_tasks"] == st0["unique_tasks"] and st2["component_dedup_hits"] == 1


def test_policy_study_modelled_time(tmp_path):
    """tools/policy_study.py (SURVEY.md §8(d) scheduler comparison) on a small repetition-heavy
    set: MICCO's modelled plan time and peer traffic do not exceed round-robin's."""
    import json
    import sys
    sys.path.insert(0, str(Path(__file__).resolve().parent.parent / "tools"))
    import policy_study
    out = tmp_path / "ps.json"
    policy_study.main(["--graphs", "300", "--N", "32", "--Lt", "8", "--rates", "0.9", "--gpus", "4",
                       "--out", str(out)])
    rows = json.loads(out.read_text())["rows"]
    for dist in ("uniform", "gaussian"):
        r = {x["policy"]: x for x in rows if x["dist"] == dist}
        assert r["micco"]["model_s"] <= r["round_robin"]["model_s"]
        assert r["micco"]["bytes_p2p"] <= r["round_robin"]["bytes_p2p"]
        assert r["micco"]["cache_hits"] >= r["round_robin"]["cache_hits"]


def test_budget_sized_window():
    """window_graphs = 0 (planner.cpp choose_window): under a budget a few rank-4
    intermediates deep, the 256-graph window spills and re-fetches, while the chosen window
    plans without any spill and with the fewest host bytes of the candidates tried; with
    room to spare the default stays one 256-graph window."""
    wl = workloads.c5_mixed(n_combos=1, Nb=8, Nm=12, Lt=2, pool=2, meson_graphs=12)
    r4 = 8 ** 4 * 2 * 16
    stats = {}
    for W in (0, 256, 64, 16):
        ctx = _ctx(mem_budget_bytes=4 * r4, window_graphs=W)
        M.load_workload(ctx, wl)
        stats[W], _ = ctx.plan(1, [0, 0, 0])
        ctx.close()
    assert stats[256]["bytes_d2h"] > 0 and stats[64]["bytes_d2h"] > 0
    assert stats[0]["bytes_d2h"] == 0 and stats[0]["evictions"] == 0
    assert stats[0]["bytes_h2d"] == min(s["bytes_h2d"] for s in stats.values())
    roomy = _ctx(mem_budget_bytes=1 << 34, window_graphs=0)
    M.load_workload(roomy, wl)
    s0, _ = roomy.plan(1, [0, 0, 0])
    roomy.close()
    fixed = _ctx(mem_budget_bytes=1 << 34, window_graphs=256)
    M.load_workload(fixed, wl)
    s256, _ = fixed.plan(1, [0, 0, 0])
    fixed.close()
    assert s0["n_stages"] == s256["n_stages"] and s0["bytes_h2d"] == s256["bytes_h2d"]


def test_affinity_policy_cuts_peer_traffic():
    """MICCO_AFFINITY (micco.h): on the weak-scaling workload (independent interleaved sets),
    preferring the operands' last consumer among Alg. 1's candidates moves fewer bytes between
    GPUs than plain MICCO, with the same balance guarantee (Alg. 1's candidate bound)."""
    wl = workloads.c2_weak_sets(4, n_graphs=1000, N=8, Lt=2, rate=0.9, seed=2)
    res = {}
    for pol in ("micco", "micco_affinity"):
        ctx = _ctx(mem_budget_bytes=1 << 30, policy=pol, window_graphs=256)
        M.load_workload(ctx, wl)
        res[pol], _ = ctx.plan(4, [1, 1, 1])
        ctx.close()
    # (0.75: repeated cycles of these r = 0.9 sets are now reused whole by canonical
    # sub-network hashing, which changes the task mix; the ratio is 0.72 with it)
    assert res["micco_affinity"]["bytes_p2p"] < 0.75 * res["micco"]["bytes_p2p"]
    assert res["micco_affinity"]["max_over_mean_load"] < 1.1
    assert res["micco_affinity"]["n_gemm"] == res["micco"]["n_gemm"]


def test_plan_model_and_demand_stats():
    """micco_plan reports the plan's window, its peak resident bytes (the memory demand C5's
    oversubscription sweep sets budgets from) and both cost-model times: copies overlapped
    (Σ_stage max_g max(flops, host, peer)) never exceeds copies serialised."""
    wl = workloads.c2_meson_set(n_graphs=200, N=16, Lt=4, rate=0.6, dist="gaussian")
    node = 16 * 16 * 4 * 16
    big = _ctx(mem_budget_bytes=1 << 40, window_graphs=32)
    M.load_workload(big, wl)
    st, _ = big.plan(2, [1, 1, 0])
    assert st["window_graphs"] == 32
    assert 0 < st["model_overlap_s"] <= st["model_s"]
    assert st["peak_bytes"] >= node and st["evictions"] == 0
    demand = st["peak_bytes"]
    tight = _ctx(mem_budget_bytes=demand // 2, window_graphs=32)
    M.load_workload(tight, wl)
    st2, _ = tight.plan(2, [1, 1, 0])
    assert st2["peak_bytes"] <= demand // 2 and st2["evictions"] > 0
    auto = _ctx(mem_budget_bytes=demand // 2)  # window_graphs = 0: sized to the budget
    M.load_workload(auto, wl)
    st3, _ = auto.plan(2, [1, 1, 0])
    assert st3["window_graphs"] >= 1 and st3["peak_bytes"] <= demand // 2


def test_set_policy_and_scalar_tables_options():
    ctx = _ctx()
    M.micco_set_policy(ctx.h, "round_robin")
    with pytest.raises(M.MiccoError):
        M.micco_set_policy(ctx.h, 9)
    M.Context(scalar_tables=1, mem_budget_bytes=1 << 30).close()
    with pytest.raises(M.MiccoError):
        M.Context(scalar_tables=2)


def test_graph_beyond_kernel_limits_rejected_at_add_graph():
    """A contraction whose slice exceeds the kernels' 32-bit per-slice offsets is refused when
    the graph is added (MICCO_ERR_UNSUPPORTED), not part-way through an execute: two N = 216
    baryons joined by one leg first (the other legs run through two mesons) give a rank-4
    intermediate with 216^4 = 2.18e9 > 2^31 elements per slice."""
    ctx = _ctx()
    N = 216
    bar = ctx.add_nodes_synth(3, N, 1, 1, [1, 2], 0, 1.0)
    mes = ctx.add_nodes_synth(2, N, 1, 1, [3, 4], 0, 1.0)
    inst = [int(bar[0]), int(bar[1]), int(mes[0]), int(mes[1])]
    edges = [(0, 0, 1, 0), (0, 1, 2, 0), (0, 2, 3, 0), (1, 1, 2, 1), (1, 2, 3, 1)]
    with pytest.raises(M.MiccoError) as e:
        ctx.add_graph(inst, edges, [0, 1, 2, 3, 4])
    assert e.value.status == -4
    ctx.close()


def test_canonical_component_reuse():
    """Canonical sub-network hashing: a connected component equal to an
    earlier one up to relabeling its instances is reused whole — cyclic rotations of a meson
    trace and reordered disconnected components; a graph with one new component is decomposed
    as usual (its known component's steps are still hash-consed); a reversed cycle is a
    different wiring (transposes) and is not reused."""
    ctx = _ctx()
    rng = np.random.default_rng(5)
    A, B, C, D, E = [ctx.add_node(rng.standard_normal((1, 4, 4)) + 0j) for _ in range(5)]
    cyc = workloads.meson_cycle_edges
    ctx.add_graph([A, B, C], cyc(3), [0, 1, 2])
    s0, _ = ctx.plan(1, [0, 0, 0])
    ctx.add_graph([B, C, A], cyc(3), [2, 0, 1])          # rotation
    ctx.add_graph([C, A, B], cyc(3), None)               # rotation, greedy order
    s1, _ = ctx.plan(1, [0, 0, 0])
    assert s1["component_dedup_hits"] == 2 and s1["unique_tasks"] == s0["unique_tasks"]
    two = [(0, 1, 1, 0), (1, 1, 0, 0), (2, 1, 3, 0), (3, 1, 2, 0)]  # tr(XY)·tr(ZW)
    ctx.add_graph([A, D, B, E], two, None)
    s2, _ = ctx.plan(1, [0, 0, 0])
    ctx.add_graph([B, E, A, D], two, None)               # the two components swapped
    s3, _ = ctx.plan(1, [0, 0, 0])
    assert s3["component_dedup_hits"] == s2["component_dedup_hits"] + 2
    assert s3["unique_tasks"] == s2["unique_tasks"]
    ctx.add_graph([A, D, C, E], two, None)               # tr(AD) known, tr(CE) new
    s4, _ = ctx.plan(1, [0, 0, 0])
    assert s4["component_dedup_hits"] == s3["component_dedup_hits"] and s4["unique_tasks"] == s3["unique_tasks"] + 1
    rev = [(0, 0, 1, 1), (1, 0, 2, 1), (2, 0, 0, 1)]      # tr(A^T B^T C^T)-style reversed wiring
    ctx.add_graph([A, B, C], rev, None)
    s5, _ = ctx.plan(1, [0, 0, 0])
    assert s5["component_dedup_hits"] == s4["component_dedup_hits"]


def test_canonical_component_reuse_large_component():
    """A 600-instance trace (edge keys past the 4096-leg range of a packed encoding) and 300
    disjoint two-meson traces: a rotation of the long trace and a reshuffle of the short ones
    are reused whole; a long trace with two neighbours swapped is a different wiring."""
    ctx = _ctx()
    rng = np.random.default_rng(9)
    ids = [ctx.add_node(rng.standard_normal((1, 2, 2)) + 0j) for _ in range(600)]
    cyc = workloads.meson_cycle_edges
    ctx.add_graph(ids, cyc(600), None)
    s0, _ = ctx.plan(1, [0, 0, 0])
    ctx.add_graph(ids[217:] + ids[:217], cyc(600), None)
    s1, _ = ctx.plan(1, [0, 0, 0])
    assert s1["component_dedup_hits"] == s0["component_dedup_hits"] + 1
    assert s1["unique_tasks"] == s0["unique_tasks"]
    sw = list(ids)
    sw[300], sw[301] = sw[301], sw[300]
    ctx.add_graph(sw, cyc(600), None)
    s2, _ = ctx.plan(1, [0, 0, 0])
    assert s2["component_dedup_hits"] == s1["component_dedup_hits"]
    pairs = [(0, 1, 1, 0), (1, 1, 0, 0)]
    inst, edges = [], []
    for i in range(300):
        inst += [ids[2 * i], ids[2 * i + 1]]
        edges += [(a + 2 * i, la, b + 2 * i, lb) for (a, la, b, lb) in pairs]
    ctx.add_graph(inst, edges, None)
    s3, _ = ctx.plan(1, [0, 0, 0])
    perm = rng.permutation(300)
    inst2 = []
    for i in perm:
        inst2 += [ids[2 * i + 1], ids[2 * i]]
    ctx.add_graph(inst2, edges, None)
    s4, _ = ctx.plan(1, [0, 0, 0])
    assert s4["component_dedup_hits"] == s3["component_dedup_hits"] + 300
    assert s4["unique_tasks"] == s3["unique_tasks"]
