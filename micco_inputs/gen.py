"""Counter-based node generator (numpy restatement of ``synth.h``) and the
workload containers.

A *node* is a hadron-node tensor T[t][i0]...[i_{r-1}] in complex double
("hadron nodes are formalized as batched matrices or
tensors", matrices for mesons, rank-3 tensors for baryons), Lt time slices,
t slowest.  A *graph* is a set of node instances whose quark legs are joined
pairwise by edges (SURVEY.md §8(c) reading #1), with
an optional reduction order (reading #8) and a complex coefficient
(reading #5).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field
from typing import List, Optional, Sequence, Tuple

import numpy as np

MODE_UNIFORM = 0
MODE_INT3 = 1

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def _splitmix64(z: np.ndarray) -> np.ndarray:
    z = z + np.uint64(0x9E3779B97F4A7C15)
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def node_scale(rank: int, N: int) -> float:
    """Entry scale s (SURVEY.md §8(c) "Value distributions"): N^-1/2 for
    mesons, N^-3/4 for baryons, written with correctly-rounded sqrt only so
    every implementation computes the identical double."""
    if rank == 2:
        return 1.0 / math.sqrt(float(N))
    if rank == 3:
        return 1.0 / math.sqrt(float(N) * math.sqrt(float(N)))
    return 1.0 / math.sqrt(float(N) ** rank)


def synth_node(seed: int, key: int, rank: int, N: int, Lt: int, mode: int = MODE_UNIFORM,
               scale: Optional[float] = None) -> np.ndarray:
    """Return the node tensor as complex128 of shape (Lt, N, ..., N); bit-identical
    to ``micco_synth_fill`` in synth.h."""
    if scale is None:
        scale = node_scale(rank, N)
    n = Lt * N ** rank
    with np.errstate(over="ignore"):
        base = _splitmix64(np.array([np.uint64(seed) ^ (np.uint64(key) * np.uint64(0xD1B54A32D192ED03))],
                                    dtype=np.uint64))[0]
        ctr = base + np.uint64(2) * np.arange(n, dtype=np.uint64)
        xr = _splitmix64(ctr)
        xi = _splitmix64(ctr + np.uint64(1))
    if mode == MODE_INT3:
        re = (xr % np.uint64(3)).astype(np.int64) - 1
        im = (xi % np.uint64(3)).astype(np.int64) - 1
        out = re.astype(np.float64) + 1j * im.astype(np.float64)
    else:
        ur = (xr >> np.uint64(11)).astype(np.float64) * 2.0 ** -53
        ui = (xi >> np.uint64(11)).astype(np.float64) * 2.0 ** -53
        out = np.empty(n, dtype=np.complex128)
        out.real = (2.0 * ur - 1.0) * scale
        out.imag = (2.0 * ui - 1.0) * scale
    return out.reshape((Lt,) + (N,) * rank)


@dataclass(frozen=True)
class NodeSpec:
    """A hadron node: rank (2 meson, 3 baryon), leg dimension N, generator key."""
    rank: int
    N: int
    key: int


Edge = Tuple[int, int, int, int]  # (u, p, v, q): leg p of instance u <-> leg q of instance v


@dataclass
class GraphSpec:
    inst: List[int]                 # node index (into Workload.nodes) per instance
    edges: List[Edge]
    order: Optional[List[int]] = None  # permutation of range(len(edges)), or None (greedy)
    coef: complex = 1.0 + 0.0j


@dataclass
class Workload:
    name: str
    Lt: int
    seed: int
    mode: int
    nodes: List[NodeSpec] = field(default_factory=list)
    graphs: List[GraphSpec] = field(default_factory=list)
    meta: dict = field(default_factory=dict)

    def node_data(self, i: int) -> np.ndarray:
        nd = self.nodes[i]
        return synth_node(self.seed, nd.key, nd.rank, nd.N, self.Lt, self.mode)

    def subset(self, graph_ids: Sequence[int], name: Optional[str] = None) -> "Workload":
        """A workload holding only the given graphs (nodes re-indexed, keys kept,
        so node tensors are unchanged)."""
        used = sorted({n for g in graph_ids for n in self.graphs[g].inst})
        remap = {old: new for new, old in enumerate(used)}
        gs = []
        for g in graph_ids:
            G = self.graphs[g]
            gs.append(GraphSpec([remap[n] for n in G.inst], list(G.edges),
                                None if G.order is None else list(G.order), G.coef))
        return Workload(name or self.name + "-subset", self.Lt, self.seed, self.mode,
                        [self.nodes[i] for i in used], gs, dict(self.meta))
