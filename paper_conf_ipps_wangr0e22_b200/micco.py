"""Thin ctypes binding of the C-ABI in include/micco.h (argument marshalling only).

Every function keeps the C name (``micco_create``, ``micco_add_hadron_node``,
``micco_add_graph``, ``micco_execute``, ``micco_get_correlator``, ...); the
``Context`` class is a convenience wrapper over them.  All computation happens
in ``libmicco.so`` (CUDA kernels for sm_100a); if the library is missing this
module raises at import of the library — there is no Python or CPU fallback.
"""
from __future__ import annotations

import ctypes
import os
from pathlib import Path
from typing import Dict, Iterable, List, Optional, Sequence, Tuple

import numpy as np

_HERE = Path(__file__).resolve().parent
LIB_PATH = _HERE / "libmicco.so"

MICCO_OK = 0
STATUS_NAMES = {0: "OK", -1: "ERR_ARG", -2: "ERR_STATE", -3: "ERR_GRAPH", -4: "ERR_UNSUPPORTED",
                -5: "ERR_OOM", -6: "ERR_CUDA", -7: "ERR_NCCL", -8: "ERR_RANGE"}
POLICIES = {"micco": 0, "micco_naive": 1, "round_robin": 2, "least_loaded": 3, "micco_affinity": 4}
SYNTH_UNIFORM, SYNTH_INT3 = 0, 1


class MiccoError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


class micco_options(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_size_t), ("mem_budget_bytes", ctypes.c_int64),
                ("policy", ctypes.c_int32), ("window_graphs", ctypes.c_int32), ("seed", ctypes.c_uint64),
                ("deterministic", ctypes.c_int32), ("keep_inputs_resident", ctypes.c_int32),
                ("dist_rank", ctypes.c_int32), ("dist_world", ctypes.c_int32), ("reorder", ctypes.c_int32),
                ("bound_model", ctypes.c_int32), ("scalar_tables", ctypes.c_int32)]


class micco_edge(ctypes.Structure):
    _fields_ = [("u", ctypes.c_int32), ("p", ctypes.c_int32), ("v", ctypes.c_int32), ("q", ctypes.c_int32)]


class micco_stats(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_size_t), ("wall_ms", ctypes.c_double), ("sched_ms", ctypes.c_double),
                ("kernel_ms", ctypes.c_double), ("copy_ms", ctypes.c_double), ("bytes_h2d", ctypes.c_int64),
                ("bytes_p2p", ctypes.c_int64), ("bytes_d2h", ctypes.c_int64), ("evictions", ctypes.c_int64),
                ("cache_hits", ctypes.c_int64), ("unique_tasks", ctypes.c_int64), ("dedup_hits", ctypes.c_int64),
                ("n_gemm", ctypes.c_int64), ("n_dot", ctypes.c_int64), ("n_stages", ctypes.c_int64),
                ("kernel_launches", ctypes.c_int64), ("flops", ctypes.c_double),
                ("flops_no_dedup", ctypes.c_double), ("max_over_mean_load", ctypes.c_double),
                ("reuse_bound", ctypes.c_int32 * 3), ("n_gpus", ctypes.c_int32),
                ("gemm_kernel_ms", ctypes.c_double), ("dot_kernel_ms", ctypes.c_double),
                ("gemm_launches", ctypes.c_int64), ("dot_launches", ctypes.c_int64),
                ("gemm_flops", ctypes.c_double), ("dot_bytes", ctypes.c_double),
                ("enqueue_ms", ctypes.c_double), ("host_pinned", ctypes.c_int32), ("gemm_3m", ctypes.c_int32),
                ("gemm_dmma_flops", ctypes.c_double), ("dot_main_ms", ctypes.c_double),
                ("dot_main_bytes", ctypes.c_double), ("dot_main_launches", ctypes.c_int64),
                ("plan_ms", ctypes.c_double), ("gemm_tma_launches", ctypes.c_int64),
                ("model_s", ctypes.c_double), ("model_overlap_s", ctypes.c_double),
                ("peak_bytes", ctypes.c_int64), ("window_graphs", ctypes.c_int32),
                ("component_dedup_hits", ctypes.c_int64), ("alloc_retries", ctypes.c_int64)]

    def as_dict(self) -> Dict:
        d = {}
        for name, _ in self._fields_:
            v = getattr(self, name)
            d[name] = list(v) if name == "reuse_bound" else v
        return d


EXPORTS = ["micco_options_default", "micco_create", "micco_destroy", "micco_add_hadron_node",
           "micco_add_hadron_nodes_synth", "micco_add_graph", "micco_execute", "micco_get_correlator",
           "micco_get_graph_value", "micco_last_error", "micco_get_stats", "micco_release_cache",
           "micco_nccl_unique_id", "micco_set_nccl_id", "micco_plan", "micco_plan_ops", "micco_dag",
           "micco_debug_schedule", "micco_plan_stages", "micco_predict_bounds", "micco_probe_fp64_peak",
           "micco_set_policy"]

_lib = None


def lib() -> ctypes.CDLL:
    """Load libmicco.so (in-tree build).  Raises if it has not been built."""
    global _lib
    if _lib is None:
        if not LIB_PATH.exists():
            raise ImportError(f"{LIB_PATH} is missing: run `python tools/build.py lib` (no CPU fallback exists)")
        L = ctypes.CDLL(str(LIB_PATH))
        P = ctypes.POINTER
        vp = ctypes.c_void_p
        L.micco_options_default.argtypes = [P(micco_options)]
        L.micco_options_default.restype = None
        L.micco_create.argtypes = [P(vp), P(micco_options)]
        L.micco_destroy.argtypes = [vp]
        L.micco_destroy.restype = None
        L.micco_add_hadron_node.argtypes = [vp, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, P(ctypes.c_double),
                                            P(ctypes.c_int64)]
        L.micco_add_hadron_nodes_synth.argtypes = [vp, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32,
                                                   ctypes.c_int32, ctypes.c_uint64, P(ctypes.c_uint64),
                                                   ctypes.c_int32, ctypes.c_double, P(ctypes.c_int64)]
        L.micco_add_graph.argtypes = [vp, ctypes.c_int32, P(ctypes.c_int64), ctypes.c_int32, P(micco_edge),
                                      P(ctypes.c_int32), ctypes.c_double, ctypes.c_double, P(ctypes.c_int64)]
        L.micco_execute.argtypes = [vp, ctypes.c_int32, P(ctypes.c_int32)]
        L.micco_get_correlator.argtypes = [vp, ctypes.c_int32, P(ctypes.c_double)]
        L.micco_get_graph_value.argtypes = [vp, ctypes.c_int64, ctypes.c_int32, P(ctypes.c_double)]
        L.micco_last_error.argtypes = [vp]
        L.micco_last_error.restype = ctypes.c_char_p
        L.micco_get_stats.argtypes = [vp, P(micco_stats)]
        L.micco_release_cache.argtypes = [vp]
        L.micco_nccl_unique_id.argtypes = [P(ctypes.c_uint8)]
        L.micco_set_nccl_id.argtypes = [vp, P(ctypes.c_uint8)]
        L.micco_plan.argtypes = [vp, ctypes.c_int32, P(ctypes.c_int32), P(micco_stats), P(ctypes.c_int32)]
        L.micco_plan_ops.argtypes = [vp, ctypes.c_int32, P(ctypes.c_int32), ctypes.c_int64, P(ctypes.c_int32),
                                     P(ctypes.c_int64), P(ctypes.c_int32)]
        L.micco_dag.argtypes = [vp, P(ctypes.c_int64), P(ctypes.c_int64), P(ctypes.c_int64), P(ctypes.c_int32),
                                P(ctypes.c_int32)]
        L.micco_debug_schedule.argtypes = [ctypes.c_int32, P(ctypes.c_int32), ctypes.c_double, ctypes.c_int32,
                                           P(ctypes.c_int64), P(ctypes.c_double), ctypes.c_int32,
                                           P(ctypes.c_int64), P(ctypes.c_int32)]
        L.micco_plan_stages.argtypes = [vp, ctypes.c_int32, ctypes.c_int32, P(ctypes.c_int32), ctypes.c_int64,
                                        P(ctypes.c_double), P(ctypes.c_int32), P(ctypes.c_int64), P(ctypes.c_double)]
        L.micco_predict_bounds.argtypes = [P(ctypes.c_double), P(ctypes.c_double), P(ctypes.c_int32)]
        L.micco_predict_bounds.restype = None
        L.micco_probe_fp64_peak.argtypes = [ctypes.c_double, P(ctypes.c_double), P(ctypes.c_double)]
        L.micco_probe_fp64_peak.restype = ctypes.c_int
        L.micco_set_policy.argtypes = [vp, ctypes.c_int32]
        for f in ("micco_set_policy", "micco_plan_stages", "micco_create", "micco_add_hadron_node", "micco_add_hadron_nodes_synth", "micco_add_graph",
                  "micco_execute", "micco_get_correlator", "micco_get_graph_value", "micco_get_stats",
                  "micco_release_cache", "micco_nccl_unique_id", "micco_set_nccl_id", "micco_plan",
                  "micco_plan_ops", "micco_dag", "micco_debug_schedule"):
            getattr(L, f).restype = ctypes.c_int
        _lib = L
    return _lib


def _ptr(a: np.ndarray, ct):
    return a.ctypes.data_as(ctypes.POINTER(ct))


def _check(ctx, st: int):
    if st != MICCO_OK:
        msg = lib().micco_last_error(ctx).decode() if ctx else ""
        raise MiccoError(st, msg)


# ---------------------------------------------------------------- C-named thin wrappers


def micco_create(mem_budget_bytes: int = 0, policy: str = "micco", window_graphs: int = 0,
                 keep_inputs_resident: bool = False, dist_rank: int = 0, dist_world: int = 0,
                 deterministic: bool = True, seed: int = 0, reorder: bool = False,
                 bound_model: int = 0, scalar_tables: int = 0) -> ctypes.c_void_p:
    o = micco_options()
    lib().micco_options_default(ctypes.byref(o))
    o.mem_budget_bytes = int(mem_budget_bytes)
    o.policy = POLICIES[policy] if isinstance(policy, str) else int(policy)
    o.window_graphs = int(window_graphs)
    o.keep_inputs_resident = 1 if keep_inputs_resident else 0
    o.dist_rank = int(dist_rank)
    o.dist_world = int(dist_world)
    o.deterministic = 1 if deterministic else 0
    o.seed = int(seed)
    o.reorder = 1 if reorder else 0
    o.bound_model = int(bound_model)
    o.scalar_tables = int(scalar_tables)
    h = ctypes.c_void_p()
    _check(None, lib().micco_create(ctypes.byref(h), ctypes.byref(o)))
    return h


def micco_destroy(ctx) -> None:
    lib().micco_destroy(ctx)


def micco_add_hadron_node(ctx, tensor: np.ndarray) -> int:
    """tensor: complex128 array of shape (Lt, N, N) or (Lt, N, N, N)."""
    a = np.ascontiguousarray(tensor, dtype=np.complex128)
    if a.ndim not in (3, 4) or any(s != a.shape[1] for s in a.shape[1:]):
        raise ValueError("node tensor must have shape (Lt, N, N) or (Lt, N, N, N)")
    out = ctypes.c_int64()
    flat = a.reshape(-1).view(np.float64)
    _check(ctx, lib().micco_add_hadron_node(ctx, a.ndim - 1, a.shape[1], a.shape[0], _ptr(flat, ctypes.c_double),
                                            ctypes.byref(out)))
    return out.value


def micco_add_hadron_nodes_synth(ctx, rank: int, N: int, Lt: int, seed: int, keys: Sequence[int], mode: int,
                                 scale: float) -> np.ndarray:
    k = np.ascontiguousarray(np.asarray(keys, dtype=np.uint64))
    ids = np.zeros(len(k), dtype=np.int64)
    _check(ctx, lib().micco_add_hadron_nodes_synth(ctx, len(k), rank, N, Lt, seed, _ptr(k, ctypes.c_uint64), mode,
                                                   scale, _ptr(ids, ctypes.c_int64)))
    return ids


def micco_add_graph(ctx, node_ids: Sequence[int], edges: Sequence[Tuple[int, int, int, int]],
                    order: Optional[Sequence[int]] = None, coef: complex = 1.0) -> int:
    nid = np.ascontiguousarray(np.asarray(node_ids, dtype=np.int64))
    E = (micco_edge * max(1, len(edges)))()
    for i, e in enumerate(edges):
        E[i] = micco_edge(*[int(x) for x in e])
    od = None
    if order is not None:
        oa = np.ascontiguousarray(np.asarray(order, dtype=np.int32))
        od = _ptr(oa, ctypes.c_int32)
    gid = ctypes.c_int64()
    coef = complex(coef)
    _check(ctx, lib().micco_add_graph(ctx, len(nid), _ptr(nid, ctypes.c_int64), len(edges), E, od, coef.real,
                                      coef.imag, ctypes.byref(gid)))
    return gid.value


def micco_execute(ctx, n_gpus: int = 1, reuse_bound: Optional[Sequence[int]] = None) -> None:
    bd = None
    if reuse_bound is not None:
        bd = (ctypes.c_int32 * 3)(*[int(x) for x in reuse_bound])
    _check(ctx, lib().micco_execute(ctx, int(n_gpus), bd))


def micco_get_correlator(ctx, t: int) -> complex:
    out = (ctypes.c_double * 2)()
    _check(ctx, lib().micco_get_correlator(ctx, int(t), out))
    return complex(out[0], out[1])


def micco_get_graph_value(ctx, graph_id: int, t: int) -> complex:
    out = (ctypes.c_double * 2)()
    _check(ctx, lib().micco_get_graph_value(ctx, int(graph_id), int(t), out))
    return complex(out[0], out[1])


def micco_get_stats(ctx) -> Dict:
    s = micco_stats()
    s.struct_size = ctypes.sizeof(micco_stats)
    _check(ctx, lib().micco_get_stats(ctx, ctypes.byref(s)))
    return s.as_dict()


def micco_release_cache(ctx) -> None:
    _check(ctx, lib().micco_release_cache(ctx))


def micco_set_policy(ctx, policy) -> None:
    _check(ctx, lib().micco_set_policy(ctx, POLICIES[policy] if isinstance(policy, str) else int(policy)))


def micco_plan(ctx, n_gpus: int, reuse_bound: Optional[Sequence[int]] = None, n_tasks: Optional[int] = None):
    s = micco_stats()
    s.struct_size = ctypes.sizeof(micco_stats)
    bd = None if reuse_bound is None else (ctypes.c_int32 * 3)(*[int(x) for x in reuse_bound])
    assign = None
    if n_tasks is not None:
        assign = np.full(max(1, n_tasks), -1, dtype=np.int32)
    _check(ctx, lib().micco_plan(ctx, int(n_gpus), bd, ctypes.byref(s),
                                 None if assign is None else _ptr(assign, ctypes.c_int32)))
    return s.as_dict(), (None if assign is None else assign[:n_tasks])


def micco_plan_ops(ctx, n_gpus: int, reuse_bound: Optional[Sequence[int]] = None):
    """(ops[n, 4] = kind, gpu, src, id in replay order; fused[task] = fused dot task or -1)."""
    bd = None if reuse_bound is None else (ctypes.c_int32 * 3)(*[int(x) for x in reuse_bound])
    n = ctypes.c_int64()
    _check(ctx, lib().micco_plan_ops(ctx, int(n_gpus), bd, 0, None, ctypes.byref(n), None))
    nt = ctypes.c_int64()
    _check(ctx, lib().micco_dag(ctx, None, ctypes.byref(nt), None, None, None))
    ops = np.zeros((max(1, n.value), 4), dtype=np.int32)
    fused = np.full(max(1, nt.value), -1, dtype=np.int32)
    _check(ctx, lib().micco_plan_ops(ctx, int(n_gpus), bd, n.value, _ptr(ops, ctypes.c_int32), ctypes.byref(n),
                                     _ptr(fused, ctypes.c_int32)))
    return ops[:n.value], fused[:nt.value]


BOUND_MODES = {"fixed": 0, "stage_sweep": 1, "regression": 2}


def micco_plan_stages(ctx, n_gpus: int, bound_mode, reuse_bound: Optional[Sequence[int]] = None):
    """(features[n_stages, 6], bounds[n_stages, 3], predicted_s) of the plan under bound_mode
    ('fixed' | 'stage_sweep' | 'regression' or 0/1/2)."""
    mode = BOUND_MODES[bound_mode] if isinstance(bound_mode, str) else int(bound_mode)
    bd = None if reuse_bound is None else (ctypes.c_int32 * 3)(*[int(x) for x in reuse_bound])
    ns, pred = ctypes.c_int64(), ctypes.c_double()
    _check(ctx, lib().micco_plan_stages(ctx, int(n_gpus), mode, bd, 0, None, None, ctypes.byref(ns),
                                        ctypes.byref(pred)))
    f = np.zeros((max(1, ns.value), 6))
    b = np.zeros((max(1, ns.value), 3), dtype=np.int32)
    _check(ctx, lib().micco_plan_stages(ctx, int(n_gpus), mode, bd, ns.value, _ptr(f, ctypes.c_double),
                                        _ptr(b, ctypes.c_int32), ctypes.byref(ns), ctypes.byref(pred)))
    return f[:ns.value], b[:ns.value], pred.value


def micco_predict_bounds(features: Sequence[float]):
    """(raw[3], bounds[3]) of the fitted reuse-bound regression on one feature vector."""
    f = np.ascontiguousarray(np.asarray(features, dtype=np.float64).reshape(6))
    raw = np.zeros(3)
    b = np.zeros(3, dtype=np.int32)
    lib().micco_predict_bounds(_ptr(f, ctypes.c_double), _ptr(raw, ctypes.c_double), _ptr(b, ctypes.c_int32))
    return raw, b


def micco_probe_fp64_peak(seconds: float = 1.0):
    """(burst, sustained) FP64 DMMA TFLOP/s of the current device (register-only loop)."""
    b, s = ctypes.c_double(), ctypes.c_double()
    st = lib().micco_probe_fp64_peak(float(seconds), ctypes.byref(b), ctypes.byref(s))
    if st != MICCO_OK:
        raise MiccoError(st, "probe_fp64_peak")
    return b.value, s.value


def micco_dag(ctx):
    """(tensor_bytes[nT], tensor_task[nT], task_info[nK, 4] = kind, a, b, out)."""
    nT, nK = ctypes.c_int64(), ctypes.c_int64()
    _check(ctx, lib().micco_dag(ctx, ctypes.byref(nT), ctypes.byref(nK), None, None, None))
    tb = np.zeros(max(1, nT.value), dtype=np.int64)
    tt = np.zeros(max(1, nT.value), dtype=np.int32)
    ti = np.zeros((max(1, nK.value), 4), dtype=np.int32)
    _check(ctx, lib().micco_dag(ctx, None, None, _ptr(tb, ctypes.c_int64), _ptr(tt, ctypes.c_int32),
                                _ptr(ti, ctypes.c_int32)))
    return tb[:nT.value], tt[:nT.value], ti[:nK.value]


def micco_nccl_unique_id() -> bytes:
    buf = (ctypes.c_uint8 * 128)()
    _check(None, lib().micco_nccl_unique_id(buf))
    return bytes(buf)


def micco_set_nccl_id(ctx, uid: bytes) -> None:
    buf = (ctypes.c_uint8 * 128)(*uid)
    _check(ctx, lib().micco_set_nccl_id(ctx, buf))


def micco_debug_schedule(n_gpus: int, reuse_bound: Sequence[int], gpu_max_memory: float,
                         vectors: Sequence[Sequence[Tuple]], resident: Iterable[Tuple[int, int]] = ()) -> List[List[int]]:
    """Native Alg. 1/2 decisions for vectors of pairs (t1, t2, out, flops, b1, b2, bout)."""
    flat = [p for v in vectors for p in v]
    off = np.zeros(len(vectors) + 1, dtype=np.int64)
    off[1:] = np.cumsum([len(v) for v in vectors])
    pairs = np.ascontiguousarray(np.asarray(flat, dtype=np.float64).reshape(-1))
    if pairs.size == 0:
        pairs = np.zeros(7)
    res_list = [tuple(r) for r in resident]
    res = np.ascontiguousarray(np.asarray(res_list, dtype=np.int64).reshape(-1))
    if res.size == 0:
        res = np.zeros(2, dtype=np.int64)
    out = np.zeros(max(1, len(flat)), dtype=np.int32)
    bd = (ctypes.c_int32 * 3)(*[int(x) for x in reuse_bound])
    st = lib().micco_debug_schedule(n_gpus, bd, float(gpu_max_memory), len(vectors), _ptr(off, ctypes.c_int64),
                                    _ptr(pairs, ctypes.c_double), len(res_list),
                                    _ptr(res, ctypes.c_int64), _ptr(out, ctypes.c_int32))
    if st != MICCO_OK:
        raise MiccoError(st, "debug_schedule")
    res_out, k = [], 0
    for v in vectors:
        res_out.append([int(x) for x in out[k:k + len(v)]])
        k += len(v)
    return res_out


# ---------------------------------------------------------------- convenience


class Context:
    """Owning wrapper over a micco_ctx."""

    def __init__(self, **kw):
        self.h = micco_create(**kw)
        self.Lt: Optional[int] = None
        self.n_graphs = 0

    def close(self):
        if self.h:
            micco_destroy(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def add_node(self, tensor: np.ndarray) -> int:
        self.Lt = tensor.shape[0]
        return micco_add_hadron_node(self.h, tensor)

    def add_nodes_synth(self, rank, N, Lt, seed, keys, mode, scale) -> np.ndarray:
        self.Lt = Lt
        return micco_add_hadron_nodes_synth(self.h, rank, N, Lt, seed, keys, mode, scale)

    def add_graph(self, node_ids, edges, order=None, coef=1.0) -> int:
        self.n_graphs += 1
        return micco_add_graph(self.h, node_ids, edges, order, coef)

    def execute(self, n_gpus=1, reuse_bound=None):
        micco_execute(self.h, n_gpus, reuse_bound)

    def correlator(self) -> np.ndarray:
        return np.array([micco_get_correlator(self.h, t) for t in range(self.Lt)], dtype=np.complex128)

    def graph_value(self, g, t) -> complex:
        return micco_get_graph_value(self.h, g, t)

    def stats(self) -> Dict:
        return micco_get_stats(self.h)

    def plan(self, n_gpus, reuse_bound=None, n_tasks=None):
        return micco_plan(self.h, n_gpus, reuse_bound, n_tasks)

    def release_cache(self):
        micco_release_cache(self.h)

    def set_policy(self, policy):
        micco_set_policy(self.h, policy)


def load_workload(ctx: Context, wl, node_arrays: Optional[Sequence[np.ndarray]] = None) -> List[int]:
    """Add a micco_inputs Workload: nodes through the synth generator (same bits as
    micco_inputs/synth.h) or explicit arrays, then every graph in order."""
    from micco_inputs.gen import node_scale  # input generation only
    ids: List[int] = [0] * len(wl.nodes)
    if node_arrays is not None:
        for i, a in enumerate(node_arrays):
            ids[i] = ctx.add_node(a)
    else:
        groups: Dict[Tuple[int, int], List[int]] = {}
        for i, nd in enumerate(wl.nodes):
            groups.setdefault((nd.rank, nd.N), []).append(i)
        for (rank, N), idx in groups.items():
            got = ctx.add_nodes_synth(rank, N, wl.Lt, wl.seed, [wl.nodes[i].key for i in idx], wl.mode,
                                      node_scale(rank, N))
            for i, nid in zip(idx, got):
                ids[i] = int(nid)
    for G in wl.graphs:
        ctx.add_graph([ids[n] for n in G.inst], G.edges, G.order, G.coef)
    ctx.Lt = wl.Lt
    return ids
