"""The seeded input generators (micco_inputs): the numpy generator agrees bit for
bit with the C header both native sides include, and the graph recipes have
the structure SURVEY.md §8(d) states."""
import collections

import numpy as np
import pytest

import oracle
from micco_inputs import workloads, synth_node
from micco_inputs.gen import MODE_INT3, MODE_UNIFORM, node_scale


@pytest.mark.parametrize("mode", [MODE_UNIFORM, MODE_INT3])
@pytest.mark.parametrize("rank,N,Lt", [(2, 5, 3), (3, 4, 2), (2, 32, 8)])
def test_numpy_generator_matches_c_header(mode, rank, N, Lt):
    wl = workloads.Workload("t", Lt, 12345, mode, [workloads.NodeSpec(rank, N, 77)], [])
    tb = oracle.NodeTable(wl)
    a = tb.tensor(0)
    b = synth_node(12345, 77, rank, N, Lt, mode)
    assert a.shape == b.shape
    assert np.array_equal(a.view(np.uint64), b.view(np.uint64))


def test_generator_ranges():
    x = synth_node(1, 2, 2, 64, 4, MODE_UNIFORM)
    s = node_scale(2, 64)
    assert np.all(np.abs(x.real) <= s) and np.all(np.abs(x.imag) <= s)
    assert abs(np.mean(x.real)) < 0.05 * s
    y = synth_node(1, 2, 3, 8, 4, MODE_INT3)
    assert set(np.unique(y.real)) == {-1.0, 0.0, 1.0}
    # different keys / seeds give different streams
    assert not np.array_equal(synth_node(1, 3, 2, 8, 2), synth_node(1, 2, 2, 8, 2))
    assert not np.array_equal(synth_node(2, 2, 2, 8, 2), synth_node(1, 2, 2, 8, 2))


def _valid_matching(wl, G):
    legs = collections.Counter()
    for (u, p, v, q) in G.edges:
        assert 0 <= p < wl.nodes[G.inst[u]].rank and 0 <= q < wl.nodes[G.inst[v]].rank
        legs[(u, p)] += 1
        legs[(v, q)] += 1
    total = sum(wl.nodes[n].rank for n in G.inst)
    assert len(legs) == total and all(c == 1 for c in legs.values())
    if G.order is not None:
        assert sorted(G.order) == list(range(len(G.edges)))


def test_c1_structure():
    wl = workloads.c1_two_meson()
    assert len(wl.graphs) == 32 and wl.Lt == 8 and all(n.N == 32 and n.rank == 2 for n in wl.nodes)
    sizes = collections.Counter(len(G.inst) for G in wl.graphs)
    assert sizes == {2: 8, 3: 8, 4: 16}
    for G in wl.graphs:
        _valid_matching(wl, G)


def test_c2_repetition_rate():
    for rate in (0.1, 0.5, 0.9):
        wl = workloads.c2_meson_set(n_graphs=2000, N=8, Lt=2, rate=rate)
        slots = sum(len(G.inst) for G in wl.graphs)
        repeated = 1.0 - len(wl.nodes) / slots
        assert abs(repeated - rate) < 0.05, (rate, repeated)
        for G in wl.graphs[:50]:
            _valid_matching(wl, G)
    g = workloads.c2_meson_set(n_graphs=2000, N=8, Lt=2, rate=0.5, dist="gaussian")
    assert len(g.graphs) == 2000


def test_c3_cycle_structure():
    wl = workloads.c3_multi_meson(n_graphs=500, N=4, Lt=2)
    for G in wl.graphs:
        _valid_matching(wl, G)
        # every edge joins a sink (0..2) and a source (3..5)
        assert all((u < 3) != (v < 3) for (u, _, v, _) in G.edges)


def test_c4_matchings():
    m = workloads.two_baryon_matchings()
    assert len(m) == 720
    # k = legs S1 shares with R1: 72 disconnected (k = 0 or 3), 648 connected
    ks = collections.Counter(sum(1 for s, r in mm if s < 3 and r < 3) for mm in m)
    assert ks[0] + ks[3] == 72 and ks[1] + ks[2] == 648
    wl = workloads.c4_two_baryon(n_combos=2, N=3, Lt=1, order="chain")
    assert len(wl.graphs) == 1440
    for G in wl.graphs[:100]:
        _valid_matching(wl, G)


def test_c5_structure():
    wl = workloads.c5_mixed(n_combos=1, Nb=3, Nm=4, Lt=1, pool=2, meson_graphs=6)
    ranks = collections.Counter(n.rank for n in wl.nodes)
    assert ranks[2] > 0 and ranks[3] > 0
    baryon = [G for G in wl.graphs if wl.nodes[G.inst[0]].rank == 3]
    assert len(baryon) == 648  # connected two-baryon matchings only
    for G in baryon[:50]:
        _valid_matching(wl, G)
        # the first contracted pair is S1 with a source sharing exactly one leg (rank-4 step)
        u, _, v, _ = G.edges[G.order[0]]
        partner = v if u == 0 else u
        shared = sum(1 for (a, _, b, _) in G.edges if {a, b} == {0, partner})
        assert shared == 1


def test_c2_weak_sets_structure():
    """bench.py's weak-scaling workload: set 0 is exactly the N = 1 C2 workload, the sets
    have disjoint node pools, and graphs are interleaved set by set."""
    from micco_inputs import workloads
    one = workloads.c2_meson_set(n_graphs=50, N=8, Lt=2, rate=0.7, seed=2)
    same = workloads.c2_weak_sets(1, n_graphs=50, N=8, Lt=2, rate=0.7, seed=2)
    assert [n.key for n in same.nodes] == [n.key for n in one.nodes]
    assert [g.inst for g in same.graphs] == [g.inst for g in one.graphs]
    assert [g.coef for g in same.graphs] == [g.coef for g in one.graphs]
    three = workloads.c2_weak_sets(3, n_graphs=50, N=8, Lt=2, rate=0.7, seed=2)
    assert len(three.graphs) == 150
    owner = {}
    for i, g in enumerate(three.graphs):
        for x in g.inst:
            assert owner.setdefault(x, i % 3) == i % 3  # graph i belongs to set i % 3
    keys = [n.key for n in three.nodes]
    assert len(set(keys)) == len(keys)
    s1 = workloads.c2_meson_set(n_graphs=50, N=8, Lt=2, rate=0.7, seed=3)
    assert [len(g.inst) for g in three.graphs[1::3]] == [len(g.inst) for g in s1.graphs]


def test_c2_weak_sets_plan_partitions():
    """Host-only plans of the 4-GPU weak-scaling workload: the MICCO scheduler finds the
    partition well enough that a repeat execute (replicas cached) moves no byte over PCIe
    and evicts nothing, while load stays balanced."""
    import os
    import paper_conf_ipps_wangr0e22_b200 as M
    from micco_inputs import workloads
    wl = workloads.c2_weak_sets(4, n_graphs=300, N=8, Lt=2, rate=0.9, seed=2)
    node_bytes = 8 * 8 * 2 * 16
    ctx = M.Context(keep_inputs_resident=True, mem_budget_bytes=400 * node_bytes, dist_rank=0, dist_world=4)
    M.load_workload(ctx, wl)
    os.environ["MICCO_PLAN_WARM"] = "1"
    try:
        st, _ = ctx.plan(4, [2, 2, 2])
    finally:
        os.environ.pop("MICCO_PLAN_WARM")
    ctx.close()
    assert st["bytes_h2d"] == 0 and st["evictions"] == 0 and st["bytes_d2h"] == 0
    assert st["max_over_mean_load"] < 1.1
