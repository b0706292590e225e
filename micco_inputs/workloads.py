"""Graph-set recipes: the synthetic workloads of SURVEY.md §8(d) (configs C1–C5
of BASELINE.json) plus small random graphs for the brute-force pins.

Every recipe is seeded (numpy PCG64) and returns a ``Workload``: node specs
(rank, N, generator key) and graphs (instances, edges, order, coefficient).
Node tensors themselves come from the counter-based generator (synth.h /
gen.synth_node), so a workload is a few KB even when its tensors are TBs.

Graph construction follows the paper's problem statement: mesons are N×N
matrices (2 quark legs), baryons N×N×N tensors (3 legs);
a graph's edges join quark legs pairwise (L11, L17); the workload knobs are
the paper's data characteristics (Table I): tensor size N, vector
size, repeated rate and Uniform/Gaussian selection of repeats (L314).
"""
from __future__ import annotations

import itertools
from typing import List, Optional, Sequence

import numpy as np

from .gen import GraphSpec, NodeSpec, Workload, MODE_UNIFORM

# ---------------------------------------------------------------- helpers


def meson_cycle_edges(k: int, flips: Optional[Sequence[bool]] = None):
    """Edges of tr(M0 M1 ... M_{k-1}) (with M_i^T where flips[i]).  Leg 0 is the
    row (quark) index, leg 1 the column (antiquark) index (SURVEY.md §8(c)
    reading #7).  Edge i joins the 'out' leg of instance i to the 'in' leg of
    instance i+1 (mod k); k == 1 is the self-edge trace."""
    flips = flips or [False] * k
    out_leg = [0 if f else 1 for f in flips]
    in_leg = [1 if f else 0 for f in flips]
    return [(i, out_leg[i], (i + 1) % k, in_leg[(i + 1) % k]) for i in range(k)]


def cycle_chain_order(n_inst: int, edges) -> List[int]:
    """Edge order that walks each cycle of a meson graph from its lowest
    instance ("chain order")."""
    at = {}
    for ei, (u, p, v, q) in enumerate(edges):
        at[(u, p)] = (ei, v, q)
        at[(v, q)] = (ei, u, p)
    seen_e, seen_u, order = set(), set(), []
    for start in range(n_inst):
        if start in seen_u:
            continue
        u, leg = start, 1
        while True:
            seen_u.add(u)
            ei, v, q = at[(u, leg)]
            if ei in seen_e:
                break
            seen_e.add(ei)
            order.append(ei)
            u, leg = v, 1 - q
    assert sorted(order) == list(range(len(edges)))
    return order


def _rand_coef(rng) -> complex:
    return complex(1.0 if rng.random() < 0.5 else -1.0, 0.0)


# ---------------------------------------------------------------- C1


def c1_two_meson(seed: int = 1, mode: int = MODE_UNIFORM, N: int = 32, Lt: int = 8,
                 pool: int = 8, per_type: int = 8) -> Workload:
    """C1 (BASELINE.json configs[0]): 32 graphs of 2–4 mesons, N=32, Lt=8.
    8 graphs each of tr(AB), tr(ABC), tr(ABCD) and tr(AB)·tr(CD); nodes drawn
    from a pool of 8 mesons, random transposes, random edge order, c_g = ±1,
    no duplicate graphs."""
    rng = np.random.default_rng(seed)
    nodes = [NodeSpec(2, N, 1000 + i) for i in range(pool)]
    graphs, seen = [], set()
    kinds = [("cyc", 2), ("cyc", 3), ("cyc", 4), ("dir", 4)]
    for kind, k in kinds:
        made = 0
        while made < per_type:
            inst = [int(x) for x in rng.integers(0, pool, size=k)]
            flips = [bool(x) for x in rng.integers(0, 2, size=k)]
            if kind == "cyc":
                edges = meson_cycle_edges(k, flips)
            else:
                e1 = meson_cycle_edges(2, flips[:2])
                e2 = [(u + 2, p, v + 2, q) for (u, p, v, q) in meson_cycle_edges(2, flips[2:])]
                edges = e1 + e2
            sig = (kind, tuple(inst), tuple(flips))
            if sig in seen:
                continue
            seen.add(sig)
            order = [int(x) for x in rng.permutation(len(edges))]
            graphs.append(GraphSpec(inst, edges, order, _rand_coef(rng)))
            made += 1
    return Workload("c1_two_meson", Lt, seed, mode, nodes, graphs, {"N": N})


# ---------------------------------------------------------------- C2


def c2_meson_set(n_graphs: int = 10000, N: int = 128, Lt: int = 64, rate: float = 0.9,
                 dist: str = "uniform", seed: int = 2, mode: int = MODE_UNIFORM,
                 flips: bool = False) -> Workload:
    """C2 (BASELINE.json configs[1]): meson-only set, each graph one cycle of
    k ∈ {3, 4} mesons, chain order.  Every node slot repeats an earlier node
    with probability `rate` (the paper's repeated rate, Table I); the
    repeated node is drawn Uniform over the nodes so far or Gaussian-biased
    toward recent ones (L314; SURVEY.md §8(c) reading #20:
    index = last − ⌊|𝒩(0, σ)|⌋, σ = max(1, pool/8))."""
    rng = np.random.default_rng(seed)
    nodes: List[NodeSpec] = []
    graphs = []
    for _ in range(n_graphs):
        k = int(rng.integers(3, 5))
        inst = []
        for _ in range(k):
            if nodes and rng.random() < rate:
                if dist == "uniform":
                    idx = int(rng.integers(0, len(nodes)))
                else:
                    sigma = max(1.0, len(nodes) / 8.0)
                    idx = len(nodes) - 1 - int(abs(rng.normal(0.0, sigma)))
                    idx = min(max(idx, 0), len(nodes) - 1)
            else:
                nodes.append(NodeSpec(2, N, 20000 + len(nodes)))
                idx = len(nodes) - 1
            inst.append(idx)
        fl = [bool(x) for x in rng.integers(0, 2, size=k)] if flips else None
        edges = meson_cycle_edges(k, fl)
        graphs.append(GraphSpec(inst, edges, cycle_chain_order(k, edges), _rand_coef(rng)))
    return Workload(f"c2_meson_set_r{rate}_{dist}", Lt, seed, mode, nodes, graphs,
                    {"N": N, "rate": rate, "dist": dist})


def c2_weak_sets(n_sets: int, n_graphs: int = 10000, N: int = 128, Lt: int = 64, rate: float = 0.9,
                 dist: str = "uniform", seed: int = 2, mode: int = MODE_UNIFORM) -> Workload:
    """Weak scaling of C2 over n_sets GPUs: n_sets independent C2 sets (seeds seed .. seed +
    n_sets − 1, disjoint node pools) in one graph stream, interleaved graph by graph.  Set 0 is
    exactly c2_meson_set(seed=seed).  The library is not told the partition: the scheduler
    must find it through operand reuse (Alg. 1)."""
    sets = [c2_meson_set(n_graphs, N, Lt, rate, dist, seed + s, mode) for s in range(n_sets)]
    nodes: List[NodeSpec] = []
    base = []
    for s, w in enumerate(sets):
        base.append(len(nodes))
        nodes += [NodeSpec(nd.rank, nd.N, nd.key + 1_000_000 * s) for nd in w.nodes]
    graphs = []
    for i in range(n_graphs):
        for s, w in enumerate(sets):
            g = w.graphs[i]
            graphs.append(GraphSpec([base[s] + x for x in g.inst], list(g.edges),
                                    None if g.order is None else list(g.order), g.coef))
    name = sets[0].name if n_sets == 1 else f"{sets[0].name}_x{n_sets}sets"
    return Workload(name, Lt, seed, mode, nodes, graphs, {"N": N, "rate": rate, "dist": dist, "sets": n_sets})


# ---------------------------------------------------------------- C3


def c3_multi_meson(n_graphs: int = 100000, N: int = 256, Lt: int = 128, pool: int = 32,
                   seed: int = 3, mode: int = MODE_UNIFORM) -> Workload:
    """C3 (configs[2]): 3-meson system.  Sinks S1..S3 from a pool, sources
    R1..R3 from a pool; each graph wires antiquark(S_a) → R_π(a) and
    quark(S_a) → R_ρ(a) for (π, ρ) ∈ S3², so cycles alternate sink/source
    (SURVEY.md §8(d) C3).  Chain order along each cycle."""
    rng = np.random.default_rng(seed)
    nodes = [NodeSpec(2, N, 30000 + i) for i in range(2 * pool)]
    perms = list(itertools.permutations(range(3)))
    graphs, seen = [], set()
    while len(graphs) < n_graphs:
        S = [int(x) for x in rng.choice(pool, 3, replace=False)]
        R = [pool + int(x) for x in rng.choice(pool, 3, replace=False)]
        pi = perms[int(rng.integers(0, 6))]
        rho = perms[int(rng.integers(0, 6))]
        sig = (tuple(S), tuple(R), pi, rho)
        if sig in seen:
            continue
        seen.add(sig)
        inst = S + R  # instances 0..2 sinks, 3..5 sources
        edges = []
        for a in range(3):
            edges.append((a, 1, 3 + pi[a], 0))   # antiquark of S_a -> R_pi(a)
            edges.append((a, 0, 3 + rho[a], 1))  # quark of S_a <- R_rho(a)
        graphs.append(GraphSpec(inst, edges, cycle_chain_order(6, edges), _rand_coef(rng)))
    return Workload("c3_multi_meson", Lt, seed, mode, nodes, graphs, {"N": N})


# ---------------------------------------------------------------- C4


def two_baryon_matchings():
    """All 720 bijections between the 6 sink legs (S1.0-2, S2.0-2) and the 6
    source legs (R1.0-2, R2.0-2), as lists of (sink_leg, source_leg) with
    legs numbered 0..5 (0-2 on the first node, 3-5 on the second)."""
    return [list(enumerate(p)) for p in itertools.permutations(range(6))]


def c4_two_baryon(n_combos: int = 64, N: int = 64, Lt: int = 64, pool: int = 8,
                  order: str = "greedy", seed: int = 4, mode: int = MODE_UNIFORM,
                  matchings: Optional[Sequence[int]] = None) -> Workload:
    """C4 (configs[3]): two-baryon correlator with rank-3 baryon tensors.
    Each graph = sinks (S1 ≠ S2), sources (R1 ≠ R2) and one of the 720
    perfect matchings of sink legs to source legs.
    order='greedy' leaves the order to the library (None); order='chain'
    contracts S1 with its 2-leg partner first (c = 2), then that partner's
    remaining leg (c = 1, rank 3), then the final rank-3 dot."""
    rng = np.random.default_rng(seed)
    nodes = [NodeSpec(3, N, 40000 + i) for i in range(2 * pool)]
    allm = two_baryon_matchings()
    msel = list(range(720)) if matchings is None else list(matchings)
    graphs, seen = [], set()
    while len(seen) < n_combos:
        S = tuple(int(x) for x in rng.choice(pool, 2, replace=False))
        R = tuple(pool + int(x) for x in rng.choice(pool, 2, replace=False))
        if (S, R) in seen:
            continue
        seen.add((S, R))
        for mi in msel:
            m = allm[mi]
            inst = [S[0], S[1], R[0], R[1]]  # instances: 0=S1, 1=S2, 2=R1, 3=R2
            edges = [(sl // 3, sl % 3, 2 + rl // 3, rl % 3) for sl, rl in m]
            od = None
            if order == "chain":
                od = _two_baryon_chain(edges)
            graphs.append(GraphSpec(inst, edges, od, _rand_coef(rng)))
    return Workload(f"c4_two_baryon_{order}", Lt, seed, mode, nodes, graphs, {"N": N})


def _two_baryon_chain(edges):
    def between(a, b):
        return [i for i, (u, _, v, _) in enumerate(edges) if {u, v} == {a, b}]
    cnt = {r: len(between(0, r)) for r in (2, 3)}
    if 2 not in cnt.values():   # disconnected (0 or 3 shared legs): any order
        return list(range(len(edges)))
    P = 2 if cnt[2] == 2 else 3
    first = between(0, P)
    second = between(P, 1)
    rest = [i for i in range(len(edges)) if i not in first and i not in second]
    return first + second + rest


# ---------------------------------------------------------------- tiny random graphs


def random_graph(rng, ranks: Sequence[int], allow_trace: bool = True, max_tries: int = 1000):
    """A random perfect matching over the legs of instances with the given ranks,
    rejecting baryon partial traces (unsupported) and keeping
    meson self-edges (traces) only when allow_trace.  Returns edges."""
    legs = [(u, p) for u, r in enumerate(ranks) for p in range(r)]
    if len(legs) % 2:
        raise ValueError("odd number of legs")
    for _ in range(max_tries):
        perm = list(rng.permutation(len(legs)))
        edges, ok = [], True
        for i in range(0, len(perm), 2):
            (u, p), (v, q) = legs[perm[i]], legs[perm[i + 1]]
            if u == v and (ranks[u] != 2 or not allow_trace):
                ok = False
                break
            edges.append((u, p, v, q))
        if ok:
            return edges
    raise RuntimeError("could not draw a valid matching")


def tiny_random(seed: int = 7, n_graphs: int = 20, N: int = 3, Lt: int = 2, mode: int = MODE_UNIFORM,
                max_inst: int = 4, baryons: bool = True) -> Workload:
    """Small random graphs (N ≤ 4, |E| ≤ 6) for the brute-force pins."""
    rng = np.random.default_rng(seed)
    nodes = [NodeSpec(2, N, 70000 + i) for i in range(4)]
    if baryons:
        nodes += [NodeSpec(3, N, 71000 + i) for i in range(4)]
    graphs = []
    while len(graphs) < n_graphs:
        n = int(rng.integers(1, max_inst + 1))
        inst = [int(x) for x in rng.integers(0, len(nodes), size=n)]
        ranks = [nodes[i].rank for i in inst]
        if sum(ranks) % 2 or sum(ranks) > 12:
            continue
        edges = random_graph(rng, ranks)
        order = [int(x) for x in rng.permutation(len(edges))]
        graphs.append(GraphSpec(inst, edges, order, _rand_coef(rng)))
    return Workload("tiny_random", Lt, seed, mode, nodes, graphs, {"N": N})


# ---------------------------------------------------------------- C5


def c5_mixed(n_combos: int = 4, Nb: int = 64, Nm: int = 256, Lt: int = 64, pool: int = 4,
             meson_graphs: int = 64, seed: int = 5, mode: int = MODE_UNIFORM) -> Workload:
    """C5 (configs[4]): memory-oversubscribed mixed meson/baryon set.

    Baryon part: connected two-baryon matchings only (S1 shares 1 or 2 legs with each
    source), with a forced first step S1 × (the source it shares exactly ONE leg with) —
    a rank-4 intermediate of Nb^4·Lt complex (16 GiB at Nb = 64, Lt = 64), shared by every
    graph with the same (S1, source, leg pair) — then that rank-4 tensor × S1's two-leg
    partner over 2 legs (rank 3), then the final rank-3 dot with S2.  Consumers of one
    rank-4 tensor are spread over the whole graph stream so it stays live.
    Meson part: C3-style 3-meson wirings at Nm, interleaved with the baryon graphs.
    Each context has one Lt (nodes may differ in N)."""
    rng = np.random.default_rng(seed)
    nodes = [NodeSpec(3, Nb, 50000 + i) for i in range(2 * pool)]
    mbase = len(nodes)
    mpool = max(3, pool)
    nodes += [NodeSpec(2, Nm, 51000 + i) for i in range(2 * mpool)]
    allm = two_baryon_matchings()
    connected = [mi for mi, m in enumerate(allm) if sum(1 for s, r in m if s < 3 and r < 3) in (1, 2)]
    baryon = []
    seen = set()
    while len(seen) < n_combos:
        S = tuple(int(x) for x in rng.choice(pool, 2, replace=False))
        R = tuple(pool + int(x) for x in rng.choice(pool, 2, replace=False))
        if (S, R) in seen:
            continue
        seen.add((S, R))
        for mi in connected:
            m = allm[mi]
            inst = [S[0], S[1], R[0], R[1]]
            edges = [(sl // 3, sl % 3, 2 + rl // 3, rl % 3) for sl, rl in m]

            def between(a, b):
                return [i for i, (u, _, v, _) in enumerate(edges) if {u, v} == {a, b}]
            one = 2 if len(between(0, 2)) == 1 else 3      # S1's single-leg partner
            two = 5 - one                                  # S1's two-leg partner
            first, second = between(0, one), between(0, two)
            rest = [i for i in range(len(edges)) if i not in first and i not in second]
            baryon.append(GraphSpec(inst, edges, first + second + rest, _rand_coef(rng)))
    rng.shuffle(baryon)
    perms = list(itertools.permutations(range(3)))
    mesons = []
    while len(mesons) < meson_graphs:
        Sm = [mbase + int(x) for x in rng.choice(mpool, 3, replace=False)]
        Rm = [mbase + mpool + int(x) for x in rng.choice(mpool, 3, replace=False)]
        pi = perms[int(rng.integers(0, 6))]
        rho = perms[int(rng.integers(0, 6))]
        edges = []
        for a in range(3):
            edges.append((a, 1, 3 + pi[a], 0))
            edges.append((a, 0, 3 + rho[a], 1))
        mesons.append(GraphSpec(Sm + Rm, edges, cycle_chain_order(6, edges), _rand_coef(rng)))
    graphs = []
    step = max(1, len(baryon) // max(1, len(mesons)))
    mi = 0
    for i, g in enumerate(baryon):
        graphs.append(g)
        if i % step == step - 1 and mi < len(mesons):
            graphs.append(mesons[mi])
            mi += 1
    graphs += mesons[mi:]
    return Workload("c5_mixed", Lt, seed, mode, nodes, graphs, {"Nb": Nb, "Nm": Nm})
