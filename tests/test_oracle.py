"""Pins for the CPU oracle (oracle/micco_oracle.c) against things other than
itself (task rule ③; SURVEY.md §8(c) "What pins each part"):

* numpy.einsum on the same index structure (a library routine implementing
  the plain definition of val_g(t));
* brute-force full index summation (O1) vs the pairwise contractor (O2);
* reduction-order invariance over ALL |E|! edge orders (|E| ≤ 6);
* closed forms: tr(I^k) = N, diagonal mesons, Levi-Civita identities
  ε·ε = 6·sign(π) and Σ_k ε_ijk ε_lmk = δ_il δ_jm − δ_im δ_jl (a rank-4
  intermediate), tr(A)tr(B) products for disconnected graphs;
* power-of-two scaling (exact) and linearity of C in c_g (exact);
* exact-integer inputs: O1 == O2 bit for bit.
A plausible mistake in O2 (dropped term, wrong sign, wrong index, transposed
operand, conjugation) changes at least one of these.
"""
import itertools
import math

import numpy as np
import pytest

import oracle
from micco_inputs import workloads
from micco_inputs.gen import GraphSpec, NodeSpec, Workload, MODE_INT3

LETTERS = "abcdefghijklmnopqrstuvwxyzABCDEFGHIJKLMNOPQRSTUVWXYZ"


def einsum_value(tensors, G, t):
    """val_g(t) via numpy.einsum: one subscript letter per edge."""
    subs = [[None] * tensors[n].ndim for n in G.inst]
    for e, (u, p, v, q) in enumerate(G.edges):
        subs[u][p - 0] = LETTERS[e]
        subs[v][q - 0] = LETTERS[e]
    ops = [tensors[n][t] for n in G.inst]
    # tensors[n] has shape (Lt, N...) so ndim includes t; subs computed on legs only
    spec = ",".join("".join(s[:tensors[n].ndim - 1]) for s, n in zip(subs, G.inst)) + "->"
    return complex(np.einsum(spec, *ops, optimize="greedy"))


def _rel(a, b):
    return abs(a - b) / max(abs(b), 1e-300)


def test_pairwise_and_brute_match_einsum_random_tiny():
    wl = workloads.tiny_random(seed=11, n_graphs=40, N=3, Lt=2)
    tb = oracle.NodeTable(wl)
    T = [tb.tensor(i) for i in range(len(wl.nodes))]
    for g in range(len(wl.graphs)):
        for t in range(wl.Lt):
            ref = einsum_value(T, wl.graphs[g], t)
            o2 = oracle.graph_value(tb, g, t)
            o2g = oracle.graph_value(tb, g, t, order="greedy")
            o1 = oracle.graph_value(tb, g, t, brute=True)
            assert _rel(o2, ref) < 1e-13 and _rel(o1, ref) < 1e-13 and _rel(o2g, ref) < 1e-13, (g, t)


def test_meson_products_vs_matmul():
    """tr(M0 M1 ... M_{k-1}) with transposes, against numpy matmul/trace."""
    rng = np.random.default_rng(5)
    N, Lt = 6, 3
    nodes = [NodeSpec(2, N, 500 + i) for i in range(5)]
    graphs = []
    for k in (1, 2, 3, 4, 5):
        for _ in range(3):
            inst = [int(x) for x in rng.integers(0, 5, size=k)]
            flips = [bool(x) for x in rng.integers(0, 2, size=k)]
            edges = workloads.meson_cycle_edges(k, flips)
            graphs.append((GraphSpec(inst, edges, [int(x) for x in rng.permutation(k)]), flips))
    wl = Workload("m", Lt, 9, 0, nodes, [g for g, _ in graphs])
    tb = oracle.NodeTable(wl)
    for gi, (G, flips) in enumerate(graphs):
        for t in range(Lt):
            M = np.eye(N, dtype=complex)
            for n, f in zip(G.inst, flips):
                A = tb.tensor(n)[t]
                M = M @ (A.T if f else A)
            assert _rel(oracle.graph_value(tb, gi, t), np.trace(M)) < 1e-13


@pytest.mark.parametrize("g", range(8))
def test_reduction_order_invariance_all_orders(g):
    """All |E|! orders give one value (SURVEY.md §8(c) 'Reduction order')."""
    wl = workloads.tiny_random(seed=21, n_graphs=8, N=2, Lt=1, max_inst=4)
    tb = oracle.NodeTable(wl)
    G = wl.graphs[g]
    ref = oracle.graph_value(tb, g, 0, brute=True)
    for perm in itertools.permutations(range(len(G.edges))):
        assert _rel(oracle.graph_value(tb, g, 0, order=list(perm)), ref) < 1e-13


def _explicit(nodes_arrays, graphs, Lt=1, name="x"):
    nodes = [NodeSpec(a.ndim - 1, a.shape[1], i) for i, a in enumerate(nodes_arrays)]
    wl = Workload(name, Lt, 0, 0, nodes, graphs)
    return wl, oracle.NodeTable(wl, arrays=nodes_arrays)


def test_identity_loops():
    N = 7
    I = np.eye(N, dtype=complex)[None]
    for k in (1, 2, 3, 4):
        wl, tb = _explicit([I], [GraphSpec([0] * k, workloads.meson_cycle_edges(k))])
        assert oracle.graph_value(tb, 0, 0) == complex(N, 0)
    # two disconnected identity loops: N * N
    e = workloads.meson_cycle_edges(2) + [(u + 2, p, v + 2, q) for (u, p, v, q) in workloads.meson_cycle_edges(2)]
    wl, tb = _explicit([I], [GraphSpec([0] * 4, e)])
    assert oracle.graph_value(tb, 0, 0) == complex(N * N, 0)


def test_diagonal_mesons():
    rng = np.random.default_rng(3)
    N = 9
    d = rng.standard_normal((3, N)) + 1j * rng.standard_normal((3, N))
    arrs = [np.diag(d[i])[None] for i in range(3)]
    wl, tb = _explicit(arrs, [GraphSpec([0, 1, 2], workloads.meson_cycle_edges(3, [False, True, False]))])
    ref = np.sum(d[0] * d[1] * d[2])
    assert _rel(oracle.graph_value(tb, 0, 0), ref) < 1e-14


def levi_civita():
    e = np.zeros((3, 3, 3), dtype=complex)
    for p in itertools.permutations(range(3)):
        sgn = np.linalg.det(np.eye(3)[list(p)])
        e[p] = round(sgn)
    return e


def _perm_sign(p):
    s = 1
    p = list(p)
    for i in range(len(p)):
        for j in range(i + 1, len(p)):
            if p[i] > p[j]:
                s = -s
    return s


def test_levi_civita_full_contraction():
    """ε_ijk ε_π(ijk) = 6·sign(π): every leg pairing of two ε baryons."""
    eps = levi_civita()[None]
    for pi in itertools.permutations(range(3)):
        edges = [(0, a, 1, pi[a]) for a in range(3)]
        for order in itertools.permutations(range(3)):
            wl, tb = _explicit([eps], [GraphSpec([0, 0], edges, list(order))])
            assert oracle.graph_value(tb, 0, 0) == complex(6 * _perm_sign(pi), 0)


def test_levi_civita_rank4_intermediate():
    """Σ_k ε_ijk ε_lmk = δ_il δ_jm − δ_im δ_jl, through a rank-4 intermediate:
    ε1·ε2 over one leg first, then against mesons A (i,l) and B (j,m) →
    tr A · tr B − tr(A B)."""
    rng = np.random.default_rng(8)
    A = rng.standard_normal((3, 3)) + 1j * rng.standard_normal((3, 3))
    B = rng.standard_normal((3, 3)) + 1j * rng.standard_normal((3, 3))
    eps = levi_civita()[None]
    # instances: 0 = ε1, 1 = ε2, 2 = A, 3 = B
    edges = [(0, 2, 1, 2), (0, 0, 2, 0), (0, 1, 3, 0), (1, 0, 2, 1), (1, 1, 3, 1)]
    wl, tb = _explicit([eps, A[None], B[None]], [GraphSpec([0, 0, 1, 2], edges, [0, 1, 2, 3, 4])])
    ref = np.trace(A) * np.trace(B) - np.trace(A @ B)
    assert _rel(oracle.graph_value(tb, 0, 0), ref) < 1e-14
    assert _rel(oracle.graph_value(tb, 0, 0, brute=True), ref) < 1e-14


def test_power_of_two_scaling_exact():
    wl = workloads.tiny_random(seed=31, n_graphs=10, N=3, Lt=2)
    tb = oracle.NodeTable(wl)
    arrays = [tb.tensor(i) * (2.0 ** (i % 3 - 1)) for i in range(len(wl.nodes))]
    tb2 = oracle.NodeTable(wl, arrays=arrays)
    for g, G in enumerate(wl.graphs):
        f = 2.0 ** sum(n % 3 - 1 for n in G.inst)
        for t in range(wl.Lt):
            assert oracle.graph_value(tb2, g, t) == oracle.graph_value(tb, g, t) * f


def test_correlator_linear_in_coefficients():
    wl = workloads.c1_two_meson(N=8, Lt=3)
    tb = oracle.NodeTable(wl)
    C, vals = oracle.correlator(wl, tb, nthreads=3, return_values=True)
    # C(t) = Σ_g c_g val_g(t), sequentially: reproduce exactly from the values
    ref = np.zeros(wl.Lt, dtype=complex)
    for g, G in enumerate(wl.graphs):
        ref = ref + G.coef * vals[g]
    assert np.array_equal(C, ref)
    for g in (0, 5, 17):
        Cg = oracle.correlator(wl, tb, nthreads=1, graph_ids=[g])
        assert np.array_equal(Cg, wl.graphs[g].coef * vals[g])
    # thread count does not change anything
    assert np.array_equal(C, oracle.correlator(wl, tb, nthreads=1))


def test_integer_mode_brute_equals_pairwise_bitwise():
    wl = workloads.tiny_random(seed=41, n_graphs=25, N=3, Lt=2, mode=MODE_INT3)
    tb = oracle.NodeTable(wl)
    for g in range(len(wl.graphs)):
        for t in range(wl.Lt):
            a = oracle.graph_value(tb, g, t)
            b = oracle.graph_value(tb, g, t, brute=True)
            assert a == b and a.real == math.floor(a.real) and a.imag == math.floor(a.imag)


def test_c1_correlator_vs_einsum():
    wl = workloads.c1_two_meson()
    tb = oracle.NodeTable(wl)
    T = [tb.tensor(i) for i in range(len(wl.nodes))]
    C = oracle.correlator(wl, tb)
    for t in range(wl.Lt):
        ref = sum(G.coef * einsum_value(T, G, t) for G in wl.graphs)
        assert _rel(C[t], ref) < 1e-12


def test_c4_two_baryon_small_orders_agree():
    """Baryon graphs (720 leg matchings) at N = 2: given chain order, greedy
    order and brute force agree (rank-3 GETT / rank-3 dot paths)."""
    wl = workloads.c4_two_baryon(n_combos=1, N=2, Lt=1, order="chain", pool=2)
    tb = oracle.NodeTable(wl)
    for g in range(0, 720, 7):
        b = oracle.graph_value(tb, g, 0, brute=True)
        assert _rel(oracle.graph_value(tb, g, 0), b) < 1e-13
        assert _rel(oracle.graph_value(tb, g, 0, order="greedy"), b) < 1e-13


def test_invalid_graphs_rejected():
    I = np.eye(2, dtype=complex)[None]
    bad = [
        [(0, 1, 1, 0)],                        # leg (0,0),(1,1) unmatched
        [(0, 1, 1, 0), (1, 1, 0, 1)],          # leg (0,1) matched twice
        [(0, 2, 1, 0), (1, 1, 0, 0)],          # leg index >= rank
    ]
    for edges in bad:
        wl, tb = _explicit([I], [GraphSpec([0, 0], edges)])
        with pytest.raises(oracle.OracleError):
            oracle.graph_value(tb, 0, 0)
