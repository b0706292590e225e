"""GPU parity: the CUDA path (through the C-ABI) against the CPU oracle on the
same seeded inputs (task rule ③).  Tolerance: ≤ 1e-10 relative per time slice
(BASELINE.json north_star); bit-exact for exact-integer inputs (SURVEY.md §8(c)
"Bit-exact GPU parity"); bitwise-identical C(t) across GPU counts, policies,
reuse bounds, windows and budgets (§8(e))."""
import numpy as np
import pytest

import oracle
import paper_conf_ipps_wangr0e22_b200 as M
from micco_inputs import workloads
from micco_inputs.gen import GraphSpec, MODE_INT3, NodeSpec, Workload

pytestmark = pytest.mark.gpu

TOL = 1e-10


def run_gpu(wl, n_gpus=1, reuse_bound=None, **kw):
    ctx = M.Context(**kw)
    M.load_workload(ctx, wl)
    ctx.execute(n_gpus, reuse_bound)
    C = ctx.correlator()
    vals = np.array([[ctx.graph_value(g, t) for t in range(wl.Lt)] for g in range(len(wl.graphs))])
    st = ctx.stats()
    ctx.close()
    return C, vals, st


def rel_err(a, b):
    return np.max(np.abs(a - b) / np.maximum(np.abs(b), 1e-300))


def check(wl, **kw):
    C, vals, st = run_gpu(wl, **kw)
    Co, valso = oracle.correlator(wl, return_values=True)
    assert rel_err(C, Co) <= TOL, (rel_err(C, Co), st)
    for g in range(len(wl.graphs)):
        assert rel_err(vals[g], valso[g]) <= TOL, g
    return C, st


def test_c1_parity():
    C, st = check(workloads.c1_two_meson())
    assert st["kernel_launches"] > 0 and st["n_gemm"] > 0


def test_c1_integer_bit_exact():
    wl = workloads.c1_two_meson(mode=MODE_INT3)
    C, vals, _ = run_gpu(wl)
    Co, valso = oracle.correlator(wl, return_values=True)
    assert np.array_equal(vals, valso)
    assert np.array_equal(C, Co)


@pytest.mark.parametrize("N", [1, 3, 33, 64, 100, 130, 257])
def test_meson_chains_ragged_shapes(N):
    """Cycles of 1..5 mesons with random transposes (all N/T operand layouts), at
    sizes that leave ragged GEMM tiles and K tails."""
    rng = np.random.default_rng(N)
    nodes = [NodeSpec(2, N, 900 + i) for i in range(5)]
    graphs = []
    for k in (1, 2, 3, 4, 5):
        for _ in range(2):
            inst = [int(x) for x in rng.integers(0, 5, size=k)]
            flips = [bool(x) for x in rng.integers(0, 2, size=k)]
            graphs.append(GraphSpec(inst, workloads.meson_cycle_edges(k, flips),
                                    [int(x) for x in rng.permutation(k)], complex(rng.choice([-1.0, 1.0]))))
    wl = Workload(f"ragged{N}", 3, 77, 0, nodes, graphs)
    check(wl)
    wl_int = Workload(f"ragged{N}i", 3, 77, MODE_INT3, nodes, graphs)
    C, vals, _ = run_gpu(wl_int)
    Co, valso = oracle.correlator(wl_int, return_values=True)
    assert np.array_equal(vals, valso)


@pytest.mark.parametrize("N", [2, 3, 5])
def test_tiny_random_graphs_with_baryons(N):
    wl = workloads.tiny_random(seed=100 + N, n_graphs=40, N=N, Lt=3)
    check(wl)
    check(wl, window_graphs=7)


@pytest.mark.parametrize("order", ["greedy", "chain"])
def test_two_baryon_all_matchings(order):
    """All 720 leg matchings of a two-baryon correlator (rank-3 GETT, c = 1 and
    c = 2, rank-3 dots with every permutation), N = 9 (ragged), Lt = 2."""
    wl = workloads.c4_two_baryon(n_combos=1, N=9, Lt=2, pool=2, order=order)
    check(wl)
    wli = workloads.c4_two_baryon(n_combos=1, N=9, Lt=2, pool=2, order=order, mode=MODE_INT3)
    C, vals, _ = run_gpu(wli)
    Co, valso = oracle.correlator(wli, return_values=True)
    assert np.array_equal(vals, valso)


@pytest.mark.parametrize("N", [4, 16])
def test_two_baryon_blocked_k(N):
    """Greedy two-baryon graphs at N = 4 and 16: every c = 2 contraction whose operands have
    no unit stride on their free or inner contracted index runs on the blocked-K GEMM
    (4 ko × 4 ki stages, kernels.cu zgemm_persistent_kb); N = 9 above leaves ragged blocks.
    Bit-exact on integer inputs."""
    wl = workloads.c4_two_baryon(n_combos=1, N=N, Lt=2, pool=2, order="greedy",
                                 matchings=list(range(0, 720, 5)))
    check(wl)
    wli = workloads.c4_two_baryon(n_combos=1, N=N, Lt=2, pool=2, order="greedy", mode=MODE_INT3,
                                  matchings=list(range(0, 720, 5)))
    C, vals, _ = run_gpu(wli)
    Co, valso = oracle.correlator(wli, return_values=True)
    assert np.array_equal(vals, valso)


def test_two_baryon_n64_sample():
    """C4 at its full tensor size (N = 64 baryons), a sample of matchings, Lt = 4."""
    wl = workloads.c4_two_baryon(n_combos=1, N=64, Lt=4, pool=2, order="chain",
                                 matchings=list(range(0, 720, 97)))
    check(wl)


def test_cross_run_invariance_bitwise():
    """C(t) is bitwise identical for any GPU count, policy, reuse bound, window and
    budget (the scalar table is exact-summed; finalize is fixed-order)."""
    wl = workloads.c2_meson_set(n_graphs=120, N=24, Lt=4, rate=0.6, dist="gaussian", flips=True)
    ref, _, _ = run_gpu(wl, 1)
    Co = oracle.correlator(wl)
    assert rel_err(ref, Co) <= TOL
    node_bytes = 24 * 24 * 4 * 16
    for n in (2, 3, 4, 8):
        for pol in ("micco", "round_robin", "least_loaded", "micco_naive", "micco_affinity"):
            C, _, _ = run_gpu(wl, n, [1, 2, 0] if pol.startswith("micco") and pol != "micco_naive" else None,
                              policy=pol, window_graphs=16)
            assert np.array_equal(C, ref), (n, pol)
    for bd in ([0, 0, 0], [2, 2, 2], None):
        C, _, _ = run_gpu(wl, 4, bd)
        assert np.array_equal(C, ref)
    for bm in (1, 2):  # per-vector bounds: sweep, regression
        C, _, _ = run_gpu(wl, 4, None, bound_model=bm, window_graphs=16)
        assert np.array_equal(C, ref), bm
    # memory pressure: evictions and host spills
    C, _, st = run_gpu(wl, 2, [1, 1, 1], mem_budget_bytes=10 * node_bytes, window_graphs=40)
    assert st["evictions"] > 0
    assert np.array_equal(C, ref)


def test_keep_inputs_resident_repeat():
    wl = workloads.c2_meson_set(n_graphs=60, N=32, Lt=4, rate=0.8)
    ctx = M.Context(keep_inputs_resident=True)
    M.load_workload(ctx, wl)
    ctx.execute(1)
    C1 = ctx.correlator()
    s1 = ctx.stats()
    ctx.execute(1)
    C2 = ctx.correlator()
    s2 = ctx.stats()
    assert np.array_equal(C1, C2)
    assert s1["bytes_h2d"] > 0 and s2["bytes_h2d"] == 0
    ctx.release_cache()
    ctx.execute(1)
    assert np.array_equal(ctx.correlator(), C1)
    ctx.close()


def test_c2_bench_config_sampled():
    """C2 at its full sizes (N = 128, Lt = 64) in the bench's launch configuration
    (windows of 256 graphs, grouped launches), 1000 graphs; 32 sampled graph values
    against the oracle computed one by one."""
    wl = workloads.c2_meson_set(n_graphs=1000, N=128, Lt=64, rate=0.9)
    ctx = M.Context()
    M.load_workload(ctx, wl)
    ctx.execute(1)
    rng = np.random.default_rng(0)
    sample = sorted(int(x) for x in rng.choice(len(wl.graphs), 32, replace=False))
    sub = wl.subset(sample)
    _, valso = oracle.correlator(sub, return_values=True)
    for i, g in enumerate(sample):
        v = np.array([ctx.graph_value(g, t) for t in range(wl.Lt)])
        assert rel_err(v, valso[i]) <= TOL, g
    ctx.close()


def test_c3_sampled_n256():
    """C3 meson wirings at N = 256 (the multi-meson config's tensor size), Lt = 4."""
    wl = workloads.c3_multi_meson(n_graphs=40, N=256, Lt=4, pool=4)
    check(wl.subset(list(range(12))))


def sampled_check(wl, n_sample, seed=0, **kw):
    """Run the whole workload through the library, then check a seeded sample of graph
    values (the oracle computes each sampled graph on its own) and the full correlator's
    consistency with the library's own per-graph values."""
    ctx = M.Context(**kw)
    M.load_workload(ctx, wl)
    ctx.execute(1)
    C = ctx.correlator()
    rng = np.random.default_rng(seed)
    sample = sorted(int(x) for x in rng.choice(len(wl.graphs), n_sample, replace=False))
    sub = wl.subset(sample)
    _, valso = oracle.correlator(sub, return_values=True)
    for i, g in enumerate(sample):
        v = np.array([ctx.graph_value(g, t) for t in range(wl.Lt)])
        assert rel_err(v, valso[i]) <= TOL, g
    vals = np.array([[ctx.graph_value(g, t) for t in range(wl.Lt)] for g in range(len(wl.graphs))])
    coefs = np.array([complex(g.coef) for g in wl.graphs])
    Csum = (coefs[:, None] * vals).sum(axis=0)
    scale = (np.abs(coefs[:, None]) * np.abs(vals)).sum(axis=0)
    assert np.max(np.abs(C - Csum) / scale) <= 1e-13
    st = ctx.stats()
    ctx.close()
    return st


def test_c3_full_size_sampled():
    """C3 at its full tensor sizes (N = 256, Lt = 128) in the bench's launch configuration
    (reuse-aware order, windows, grouped 3M launches with the fused final dot): 300 graphs,
    32 sampled graph values against the oracle computed graph by graph."""
    wl = workloads.c3_multi_meson(n_graphs=300, N=256, Lt=128, pool=6)
    st = sampled_check(wl, 32, reorder=True)
    assert st["n_gemm"] > 0


def test_c4_full_size_sampled():
    """C4 at its full sizes (N = 64 rank-3 baryons, Lt = 64) in the bench's launch
    configuration (greedy order: c = 2 GETTs with K = 4096 on the persistent and blocked-K
    kernels, then 64×64 dots): one sink/source combination's 720 matchings, 32 sampled."""
    wl = workloads.c4_two_baryon(n_combos=1, N=64, Lt=64, pool=2, order="greedy")
    st = sampled_check(wl, 32, seed=1)
    assert st["n_gemm"] > 0


def test_multiprocess_mode_single_rank_nccl():
    """The one-process-per-GPU path (plan replay of this rank's ops, NCCL communicator,
    ncclAllReduce of the scalar table) with world size 1: same C(t) bit for bit."""
    wl = workloads.c1_two_meson()
    ref, _, _ = run_gpu(wl)
    ctx = M.Context(dist_rank=0, dist_world=1)
    M.load_workload(ctx, wl)
    M.micco_set_nccl_id(ctx.h, M.micco_nccl_unique_id())
    ctx.execute(1)
    C = ctx.correlator()
    ctx.close()
    assert np.array_equal(C, ref)


def test_c5_mixed_oversubscribed():
    """C5 shape, scaled down: rank-4 baryon intermediates (forced c = 1 first step) mixed
    with 3-meson graphs (different N in one context), on 2 logical GPUs with a budget a
    few rank-4 tensors deep — evictions, D2H spills and peer copies — against the oracle."""
    wl = workloads.c5_mixed(n_combos=1, Nb=6, Nm=10, Lt=2, pool=2, meson_graphs=12)
    r4_bytes = 6 ** 4 * 2 * 16
    C, vals, st = run_gpu(wl, 2, [1, 1, 1], mem_budget_bytes=2 * r4_bytes, window_graphs=32)
    Co, valso = oracle.correlator(wl, return_values=True)
    assert rel_err(C, Co) <= TOL
    assert st["evictions"] > 0 and st["bytes_d2h"] > 0 and st["bytes_p2p"] > 0, st
    ref, _, _ = run_gpu(wl, 1)
    assert np.array_equal(C, ref)


def test_reorder_parity():
    """Reuse-aware reduction order (options.reorder): the caller's
    order is replaced, the values are not — against the oracle (which contracts in the
    caller's order) on C3 wirings, random meson/baryon graphs and C4 chain graphs, bit-exact
    on integer inputs, and bitwise identical across GPU counts."""
    check(workloads.c3_multi_meson(n_graphs=60, N=40, Lt=3, pool=4), reorder=True)
    check(workloads.tiny_random(seed=7, n_graphs=40, N=3, Lt=2), reorder=True)
    check(workloads.c4_two_baryon(n_combos=1, N=9, Lt=2, pool=2, order="chain"), reorder=True)
    wli = workloads.c3_multi_meson(n_graphs=60, N=40, Lt=2, pool=4, mode=MODE_INT3)
    _, vals, _ = run_gpu(wli, reorder=True)
    _, valso = oracle.correlator(wli, return_values=True)
    assert np.array_equal(vals, valso)
    wl = workloads.c2_meson_set(n_graphs=120, N=24, Lt=4, rate=0.6, dist="gaussian", flips=True)
    ref, _, _ = run_gpu(wl, 1, reorder=True)
    assert rel_err(ref, oracle.correlator(wl)) <= TOL
    for n in (2, 4):
        C, _, _ = run_gpu(wl, n, [1, 2, 0], reorder=True, window_graphs=16)
        assert np.array_equal(C, ref), n


def test_streamed_planning_bitwise(monkeypatch):
    """Streamed planning (executor.cu PlanStream: the planner thread publishes each stage's
    ops while earlier stages are replayed) gives the same C(t), bit for bit, as replaying a
    finished plan — on 1 and 3 logical GPUs, with cached and with released node replicas."""
    wl = workloads.c3_multi_meson(n_graphs=80, N=40, Lt=3, pool=4)
    Co = oracle.correlator(wl)
    for n in (1, 3):
        res = {}
        for mode in ("0", "1"):
            monkeypatch.setenv("MICCO_NO_PLAN_STREAM", mode)
            ctx = M.Context(keep_inputs_resident=True, window_graphs=8)
            M.load_workload(ctx, wl)
            out = []
            for rep in range(3):  # first execute plans synchronously; later ones stream
                if rep == 2:
                    ctx.release_cache()
                ctx.execute(n, [1, 1, 0] if n > 1 else None)
                out.append(ctx.correlator())
            ctx.close()
            res[mode] = out
        for a, b in zip(res["0"], res["1"]):
            assert np.array_equal(a, b), n
        assert rel_err(res["0"][-1], Co) <= TOL


def test_gpu_count_change_in_one_context():
    """One context executed on 2, then 1, then 3 logical GPUs (each switch tears the executor
    down and sets it up again): the same C(t) bit for bit, and graph values readable after
    each.  (Regression: the per-graph value table was not reallocated after a re-setup.)"""
    wl = workloads.c2_meson_set(n_graphs=90, N=24, Lt=3, rate=0.7)
    ctx = M.Context(keep_inputs_resident=True)
    M.load_workload(ctx, wl)
    out = []
    for n in (2, 1, 3, 1):
        ctx.execute(n)
        out.append(ctx.correlator())
        assert np.isfinite(ctx.graph_value(len(wl.graphs) - 1, 2))
    ctx.close()
    for C in out[1:]:
        assert np.array_equal(C, out[0])
    assert rel_err(out[0], oracle.correlator(wl)) <= TOL


# ---------------------------------------------------------------- round-2 parity additions


def test_add_hadron_node_with_caller_arrays():
    """The paper's interface with caller-owned buffers (hadron nodes as batched
    matrices / tensors; include/micco.h micco_add_hadron_node): C1 and a C4 sample built from
    explicit complex128 arrays, not the synth extension.  Same C(t) as the oracle (≤ 1e-10),
    bit-exact on integer inputs, bitwise equal to the synth-loaded run, and identical content
    is deduplicated to one node id."""
    for wl in (workloads.c1_two_meson(),
               workloads.c4_two_baryon(n_combos=1, N=16, Lt=4, pool=2, order="greedy",
                                       matchings=list(range(0, 720, 7)))):
        arrays = [wl.node_data(i) for i in range(len(wl.nodes))]
        ctx = M.Context()
        ids = M.load_workload(ctx, wl, node_arrays=arrays)
        assert len(set(ids)) == len(ids)
        assert ctx.add_node(arrays[0].copy()) == ids[0]  # content dedup (hash + memcmp)
        ctx.execute(1)
        C = ctx.correlator()
        vals = np.array([[ctx.graph_value(g, t) for t in range(wl.Lt)] for g in range(len(wl.graphs))])
        ctx.close()
        Co, valso = oracle.correlator(wl, return_values=True)
        assert rel_err(C, Co) <= TOL, wl.name
        for g in range(len(wl.graphs)):
            assert rel_err(vals[g], valso[g]) <= TOL, (wl.name, g)
        Cs, _, _ = run_gpu(wl)
        assert np.array_equal(C, Cs), wl.name
    wli = workloads.c1_two_meson(mode=MODE_INT3)
    ctx = M.Context()
    M.load_workload(ctx, wli, node_arrays=[wli.node_data(i) for i in range(len(wli.nodes))])
    ctx.execute(1)
    vals = np.array([[ctx.graph_value(g, t) for t in range(wli.Lt)] for g in range(len(wli.graphs))])
    ctx.close()
    _, valso = oracle.correlator(wli, return_values=True)
    assert np.array_equal(vals, valso)


def _n_components(G):
    parent = list(range(len(G.inst)))

    def find(x):
        while parent[x] != x:
            x = parent[x]
        return x
    for u, _, v, _ in G.edges:
        parent[find(u)] = find(v)
    return len({find(i) for i in range(len(G.inst))})


@pytest.mark.parametrize("reorder", [False, True])
def test_c3_six_cycle_integer_bit_exact_n256(reorder):
    """Full-size (N = 256) C3 six-meson cycles on exact-integer inputs (re, im ∈ {−1, 0, 1}):
    every partial sum is an integer below N^6·2^3 ≈ 2.3e15 < 2^53, so the GPU's 3M DMMA
    GEMM chain plus the fused final dot must reproduce the oracle bit for bit
    (SURVEY.md §8(c) "Bit-exact GPU parity")."""
    wl = workloads.c3_multi_meson(n_graphs=60, N=256, Lt=2, pool=4, mode=MODE_INT3)
    six = [g for g, G in enumerate(wl.graphs) if _n_components(G) == 1][:8]
    assert len(six) >= 4
    sub = wl.subset(six)
    _, vals, st = run_gpu(sub, reorder=reorder)
    _, valso = oracle.correlator(sub, return_values=True)
    assert st["n_gemm"] > 0
    assert np.array_equal(vals, valso)
    assert np.max(np.abs(valso)) > 2.0 ** 20  # sums of ~2.8e14 integer terms


def test_rank4_parity_nb64():
    """C5's rank-4 path at its stated baryon size, Nb = 64 (intermediates need
    significant memory): S1 × R over one leg → a 64^4 rank-4 intermediate per slice
    (16.7 M complex), then rank-4 × rank-3 over two legs, then the rank-3 dot.  Lt = 2 keeps
    the oracle at ~9 GFLOP per graph; the whole set runs on the GPU and 3 baryon graphs plus
    one meson graph are checked against the oracle one by one."""
    wl = workloads.c5_mixed(n_combos=1, Nb=64, Nm=64, Lt=2, pool=2, meson_graphs=4)
    ctx = M.Context()
    M.load_workload(ctx, wl)
    ctx.execute(1)
    bary = [g for g, G in enumerate(wl.graphs) if wl.nodes[G.inst[0]].rank == 3]
    mes = [g for g, G in enumerate(wl.graphs) if wl.nodes[G.inst[0]].rank == 2]
    rng = np.random.default_rng(4)
    sample = sorted([int(x) for x in rng.choice(bary, 3, replace=False)] + [mes[0]])
    _, valso = oracle.correlator(wl.subset(sample), return_values=True)
    for i, g in enumerate(sample):
        v = np.array([ctx.graph_value(g, t) for t in range(wl.Lt)])
        assert rel_err(v, valso[i]) <= TOL, g
    st = ctx.stats()
    ctx.close()
    assert st["n_gemm"] > 0


@pytest.mark.parametrize("tma", ["1", "0"])
def test_gemm_paths_meson_shapes(tma, monkeypatch):
    """Both GEMM kernels on the meson shapes the TMA kernel takes (MICCO_GEMM_TMA=0 keeps every
    contraction on the cp.async persistent kernel, which otherwise serves only ragged / strided
    operands): C2 cycles with random transposes (all four operand-layout classes) and C3 wirings
    with the reuse-aware order (fused final dots), ≤ 1e-10 against the oracle, and integer
    inputs bit-exact; the TMA run must really use the TMA kernel."""
    monkeypatch.setenv("MICCO_GEMM_TMA", tma)
    for wl in (workloads.c2_meson_set(n_graphs=60, N=128, Lt=3, rate=0.5, flips=True),
               workloads.c3_multi_meson(n_graphs=40, N=128, Lt=2, pool=4)):
        C, st = check(wl, reorder=True)
        assert (st["gemm_tma_launches"] > 0) == (tma == "1"), st
        assert st["gemm_tma_launches"] <= st["gemm_launches"]
    wli = workloads.c2_meson_set(n_graphs=40, N=128, Lt=2, rate=0.5, flips=True, mode=MODE_INT3)
    _, vals, _ = run_gpu(wli)
    _, valso = oracle.correlator(wli, return_values=True)
    assert np.array_equal(vals, valso)


def test_tma_gemm_ragged_tiles():
    """The TMA kernel's zero-filled boxes: meson cycles at N = 1032 (the smallest N above 1024
    whose 128-row tiles it takes: 1032 = 8·128 + 8 rows, 32·32 + 8 columns, k = 64·16 + 8), so
    every tile edge and the last k-stage are ragged; all four operand-layout classes via random
    transposes; ≤ 1e-10 against the oracle and the TMA kernel really used."""
    rng = np.random.default_rng(5)
    N = 1032
    nodes = [NodeSpec(2, N, 700 + i) for i in range(3)]
    graphs = []
    for k in (2, 3, 3, 2):
        inst = [int(x) for x in rng.integers(0, 3, size=k)]
        flips = [bool(x) for x in rng.integers(0, 2, size=k)]
        graphs.append(GraphSpec(inst, workloads.meson_cycle_edges(k, flips), list(range(k)),
                                complex(rng.choice([-1.0, 1.0]))))
    wl = Workload("ragged1032", 1, 91, 0, nodes, graphs)
    C, st = check(wl)
    assert st["gemm_tma_launches"] > 0, st


def test_shared_operand_dot_groups():
    """The shared-operand dot kernel (kernels.cu zdot_group_kernel): greedy two-baryon graphs at
    N = 16 (every final dot is a 16 × 16 flat or transposed dot; the c = 2 products are the A side
    of many dots, so groups fill up to kDotGroupPartners and batches split them), against the
    oracle, integer inputs bit-exact, and every graph value bitwise the same under other
    groupings (windows, GPU counts, per-GPU tables); plus meson cycles at N = 64 (the largest
    groupable slice) and 65 (the CTA dot kernel) against the oracle."""
    wl = workloads.c4_two_baryon(n_combos=1, N=16, Lt=3, pool=2, order="greedy")
    C, vals, st = run_gpu(wl)
    Co, valso = oracle.correlator(wl, return_values=True)
    assert rel_err(C, Co) <= TOL
    for g in range(len(wl.graphs)):
        assert rel_err(vals[g], valso[g]) <= TOL, g
    for kw in ({"window_graphs": 7}, {"window_graphs": 300}, {"n_gpus": 3, "scalar_tables": 1}):
        n = kw.pop("n_gpus", 1)
        C2, vals2, _ = run_gpu(wl, n, **kw)
        assert np.array_equal(vals2, vals), kw
        assert np.array_equal(C2, C), kw
    wli = workloads.c4_two_baryon(n_combos=1, N=16, Lt=2, pool=2, order="greedy", mode=MODE_INT3,
                                  matchings=list(range(0, 720, 3)))
    _, vals, _ = run_gpu(wli)
    _, valso = oracle.correlator(wli, return_values=True)
    assert np.array_equal(vals, valso)
    for N in (64, 65):
        rng = np.random.default_rng(N)
        nodes = [NodeSpec(2, N, 300 + i) for i in range(3)]
        graphs = []
        for k in (2, 2, 3, 4, 4):
            inst = [int(x) for x in rng.integers(0, 3, size=k)]
            flips = [bool(x) for x in rng.integers(0, 2, size=k)]
            graphs.append(GraphSpec(inst, workloads.meson_cycle_edges(k, flips), list(range(k)),
                                    complex(rng.choice([-1.0, 1.0]))))
        check(Workload(f"dots{N}", 2, 5 + N, 0, nodes, graphs))


def test_repeat_bitwise_at_scale():
    """Bitwise reproducibility of every graph value over repeated executes and fresh contexts at
    C3's tensor size (N = 256, Lt = 128, 2000 graphs, reuse-aware order: TMA GEMMs with fused
    dots).  Guards the TMA ring's slot release: without the proxy fence before the consumers'
    empty-barrier arrive, a TMA write could overtake queued LDS of the slot it refills (about one
    wrong (graph, slice) per 20 executes of 10k graphs; tools/race_hunt.py)."""
    wl = workloads.c3_multi_meson(n_graphs=2000, N=256, Lt=128)
    ref = None
    for _ in range(2):
        ctx = M.Context(keep_inputs_resident=True, reorder=True)
        M.load_workload(ctx, wl)
        for _ in range(3):
            ctx.execute(1)
            st = ctx.stats()
            assert st["gemm_tma_launches"] > 0
            vals = np.array([[ctx.graph_value(g, t) for t in range(wl.Lt)] for g in range(len(wl.graphs))])
            if ref is None:
                ref = vals
            else:
                bad = np.argwhere(vals != ref)
                assert len(bad) == 0, bad[:10]
        ctx.close()


def test_canonical_component_reuse_parity():
    """Graphs that repeat earlier ones up to instance relabeling (a random permutation of
    the instances with the edges remapped, and their own random reduction orders) reuse the
    earlier components' scalars (component_dedup_hits); every graph value still matches the
    oracle, which contracts each graph on its own in its own order (≤ 1e-10; bit-exact on
    integer inputs)."""
    for mode in (0, MODE_INT3):
        base = workloads.c1_two_meson(mode=mode)
        rng = np.random.default_rng(11)
        graphs = list(base.graphs)
        for G in base.graphs[:24]:
            n = len(G.inst)
            p = [int(x) for x in rng.permutation(n)]  # old instance i -> new label p[i]
            inst = [None] * n
            for i in range(n):
                inst[p[i]] = G.inst[i]
            edges = [(p[a], la, p[b], lb) for (a, la, b, lb) in G.edges]
            graphs.append(GraphSpec(inst, edges, [int(x) for x in rng.permutation(len(edges))], G.coef))
        wl = Workload(base.name + "-perm", base.Lt, base.seed, base.mode, base.nodes, graphs)
        C, vals, st = run_gpu(wl)
        assert st["component_dedup_hits"] > 0, st
        Co, valso = oracle.correlator(wl, return_values=True)
        if mode == MODE_INT3:
            assert np.array_equal(vals, valso)
        else:
            assert rel_err(C, Co) <= TOL
            for g in range(len(graphs)):
                assert rel_err(vals[g], valso[g]) <= TOL, g
