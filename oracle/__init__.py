"""CPU ORACLE — test infrastructure only.

Plain, slow, obviously-correct CPU implementations of what the MICCO hot path
computes, used to pin the CUDA library (task rule ③):

* ``liboracle.so`` (micco_oracle.c): brute-force index summation (O1) and the
  naive pairwise contractor (O2) for graph values, and the correlator
  C(t) = Σ_g c_g val_g(t).
* ``sched.py``: the paper's scheduler, Alg. 1 + Alg. 2, restated line by line
  (PAPER.md L203-288).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  It shares no code with
``paper_conf_ipps_wangr0e22_b200`` and imports nothing from it; the only common
source is the input generator ``micco_inputs``.
"""
from __future__ import annotations

import ctypes
import os
from pathlib import Path
from typing import List, Optional, Sequence

import numpy as np

_HERE = Path(__file__).resolve().parent
_LIB = None


class _Node(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_int32), ("N", ctypes.c_int32), ("data", ctypes.POINTER(ctypes.c_double))]


class _Edge(ctypes.Structure):
    _fields_ = [("u", ctypes.c_int32), ("p", ctypes.c_int32), ("v", ctypes.c_int32), ("q", ctypes.c_int32)]


def lib():
    global _LIB
    if _LIB is None:
        so = _HERE / "liboracle.so"
        if not so.exists():
            import sys
            sys.path.insert(0, str(_HERE.parent / "tools"))
            from build import build_oracle  # type: ignore
            build_oracle()
        L = ctypes.CDLL(str(so))
        dp = ctypes.POINTER(ctypes.c_double)
        ip = ctypes.POINTER(ctypes.c_int32)
        L.orc_graph_value.argtypes = [ctypes.POINTER(_Node), ctypes.c_int32, ctypes.c_int32, ip, ctypes.c_int32,
                                      ctypes.POINTER(_Edge), ip, ctypes.c_int32, dp]
        L.orc_graph_value_brute.argtypes = [ctypes.POINTER(_Node), ctypes.c_int32, ctypes.c_int32, ip,
                                            ctypes.c_int32, ctypes.POINTER(_Edge), ctypes.c_int32, dp]
        L.orc_correlator.argtypes = [ctypes.POINTER(_Node), ctypes.c_int32, ctypes.c_int32, ip, ip, ip,
                                     ctypes.POINTER(_Edge), ip, ip, dp, ctypes.c_int32, dp, dp]
        L.orc_synth_node.argtypes = [dp, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int64, ctypes.c_int32,
                                     ctypes.c_double]
        for f in (L.orc_graph_value, L.orc_graph_value_brute, L.orc_correlator):
            f.restype = ctypes.c_int
        L.orc_synth_node.restype = None
        _LIB = L
    return _LIB


class OracleError(RuntimeError):
    pass


def _check(rc):
    if rc != 0:
        raise OracleError(f"oracle returned status {rc}")


def _i32(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.int32))


class NodeTable:
    """Node tensors for the oracle, as interleaved float64 buffers (the C-ABI
    layout).  Filled from the shared generator (micco_inputs/synth.h) through
    ``orc_synth_node``, or from explicit complex arrays."""

    def __init__(self, workload, arrays: Optional[Sequence[np.ndarray]] = None):
        from micco_inputs.gen import node_scale
        self.wl = workload
        self.bufs: List[np.ndarray] = []
        for i, nd in enumerate(workload.nodes):
            n = workload.Lt * nd.N ** nd.rank
            if arrays is not None:
                a = np.ascontiguousarray(np.asarray(arrays[i], dtype=np.complex128)).reshape(-1)
                if a.size != n:
                    raise ValueError("node array has the wrong size")
                buf = a.view(np.float64).copy()
            else:
                buf = np.empty(2 * n, dtype=np.float64)
                lib().orc_synth_node(buf.ctypes.data_as(ctypes.POINTER(ctypes.c_double)), workload.seed, nd.key,
                                     n, workload.mode, node_scale(nd.rank, nd.N))
            self.bufs.append(buf)
        self.c_nodes = (_Node * max(1, len(self.bufs)))()
        for i, (nd, b) in enumerate(zip(workload.nodes, self.bufs)):
            self.c_nodes[i] = _Node(nd.rank, nd.N, b.ctypes.data_as(ctypes.POINTER(ctypes.c_double)))

    def tensor(self, i: int) -> np.ndarray:
        nd = self.wl.nodes[i]
        return self.bufs[i].view(np.complex128).reshape((self.wl.Lt,) + (nd.N,) * nd.rank)


def _edges(edges) -> ctypes.Array:
    arr = (_Edge * max(1, len(edges)))()
    for i, e in enumerate(edges):
        arr[i] = _Edge(*[int(x) for x in e])
    return arr


def graph_value(table: NodeTable, g: int, t: int, order="given", brute: bool = False) -> complex:
    """val_g(t) by O2 (pairwise, along `order`: 'given', 'greedy' or a list) or O1."""
    G = table.wl.graphs[g]
    inst = _i32(G.inst)
    ed = _edges(G.edges)
    out = (ctypes.c_double * 2)()
    ip = ctypes.POINTER(ctypes.c_int32)
    if brute:
        _check(lib().orc_graph_value_brute(table.c_nodes, table.wl.Lt, len(G.inst), inst.ctypes.data_as(ip),
                                           len(G.edges), ed, t, out))
    else:
        if isinstance(order, str):
            od = None if (order == "greedy" or G.order is None) else _i32(G.order)
        else:
            od = _i32(order)
        _check(lib().orc_graph_value(table.c_nodes, table.wl.Lt, len(G.inst), inst.ctypes.data_as(ip),
                                     len(G.edges), ed, None if od is None else od.ctypes.data_as(ip), t, out))
    return complex(out[0], out[1])


def correlator(workload, table: Optional[NodeTable] = None, nthreads: Optional[int] = None,
               graph_ids: Optional[Sequence[int]] = None, return_values: bool = False):
    """C(t), t = 0..Lt-1, as complex128 (and optionally val_g(t) as [G, Lt])."""
    table = table or NodeTable(workload)
    gids = list(range(len(workload.graphs))) if graph_ids is None else list(graph_ids)
    inst_off, inst, edge_off, edges, orders, has_order, coefs = [0], [], [0], [], [], [], []
    for g in gids:
        G = workload.graphs[g]
        inst += list(G.inst)
        inst_off.append(len(inst))
        edges += list(G.edges)
        orders += list(G.order) if G.order is not None else [0] * len(G.edges)
        has_order.append(0 if G.order is None else 1)
        edge_off.append(len(edges))
        coefs += [G.coef.real, G.coef.imag]
    ip = ctypes.POINTER(ctypes.c_int32)
    dp = ctypes.POINTER(ctypes.c_double)
    a_io, a_in, a_eo, a_or, a_ho = (_i32(x) for x in (inst_off, inst, edge_off, orders or [0], has_order or [0]))
    a_cf = np.ascontiguousarray(np.asarray(coefs or [0.0], dtype=np.float64))
    Lt = workload.Lt
    vals = np.zeros((len(gids), Lt, 2), dtype=np.float64)
    corr = np.zeros((Lt, 2), dtype=np.float64)
    nt = nthreads or os.cpu_count() or 1
    _check(lib().orc_correlator(table.c_nodes, Lt, len(gids), a_io.ctypes.data_as(ip), a_in.ctypes.data_as(ip),
                                a_eo.ctypes.data_as(ip), _edges(edges), a_or.ctypes.data_as(ip),
                                a_ho.ctypes.data_as(ip), a_cf.ctypes.data_as(dp), nt, vals.ctypes.data_as(dp),
                                corr.ctypes.data_as(dp)))
    c = corr[:, 0] + 1j * corr[:, 1]
    if return_values:
        return c, vals[..., 0] + 1j * vals[..., 1]
    return c
