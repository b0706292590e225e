"""The cross-GPU data plane (north_star "final cross-GPU NCCL
reduce"): per-GPU scalar tables summed exactly, NVLink peer moves, and the one-process-per-GPU
path with ncclSend/ncclRecv of intermediates plus the ncclAllReduce of the scalar tables.

* `scalar_tables = 1` gives every logical GPU its own table, so the combine (copy of each
  table to the home GPU + exact accumulate) runs on one B200: C(t) must be bitwise equal to
  the one-table run and to 1 GPU, and within 1e-10 of the oracle (a stage's
  pairs run on different GPUs; every slot is nonzero in exactly one table).
* With two or more CUDA devices: the single-process multi-device path (cudaMemcpyPeerAsync
  between devices, pool peer access) and the multi-process NCCL path at world size 2 (spawned
  processes, one per GPU).  On a one-GPU box these are collected and skipped.
"""
import os
import socket

import numpy as np
import pytest
import torch

import oracle
import paper_conf_ipps_wangr0e22_b200 as M
from micco_inputs import workloads

pytestmark = pytest.mark.gpu

TOL = 1e-10


def rel_err(a, b):
    return np.max(np.abs(a - b) / np.maximum(np.abs(b), 1e-300))


def run(wl, n, bd=None, **kw):
    ctx = M.Context(**kw)
    M.load_workload(ctx, wl)
    ctx.execute(n, bd)
    C = ctx.correlator()
    vals = np.array([[ctx.graph_value(g, t) for t in range(wl.Lt)] for g in range(len(wl.graphs))])
    st = ctx.stats()
    ctx.close()
    return C, vals, st


def c5_small():
    """C5 shape scaled down: rank-4 baryon intermediates (forced c = 1 first step) mixed with
    meson graphs; with a budget two rank-4 tensors deep it evicts, spills and peer-copies."""
    return workloads.c5_mixed(n_combos=1, Nb=6, Nm=10, Lt=2, pool=2, meson_graphs=12)


C5_KW = dict(mem_budget_bytes=2 * 6 ** 4 * 2 * 16, window_graphs=32)


def test_per_gpu_scalar_tables_combine():
    """2, 3 and 8 logical GPUs, each with its own scalar table: the combine runs (one
    accumulate launch per extra table) and C(t) is bitwise the 1-GPU result."""
    wl = workloads.c2_meson_set(n_graphs=120, N=24, Lt=4, rate=0.6, dist="gaussian", flips=True)
    Co, valso = oracle.correlator(wl, return_values=True)
    ref, ref_vals, _ = run(wl, 1)
    assert rel_err(ref, Co) <= TOL
    for n in (2, 3, 8):
        C0, _, s0 = run(wl, n, [1, 2, 0], window_graphs=16)
        C1, vals1, s1 = run(wl, n, [1, 2, 0], window_graphs=16, scalar_tables=1)
        assert s1["kernel_launches"] - s0["kernel_launches"] == n - 1, (n, s0, s1)
        assert np.array_equal(C1, ref), n
        assert np.array_equal(C0, ref), n
        assert np.array_equal(vals1, ref_vals), n
        assert rel_err(C1, Co) <= TOL


def test_per_gpu_scalar_tables_with_evictions_and_peer_copies():
    """C5-small on 2 and 4 logical GPUs with separate tables, evictions, spills and peer
    copies: within 1e-10 of the oracle and bitwise equal to 1 GPU."""
    wl = c5_small()
    Co = oracle.correlator(wl)
    ref, _, _ = run(wl, 1)
    for n in (2, 4):
        C, _, st = run(wl, n, [1, 1, 1], scalar_tables=1, **C5_KW)
        assert st["evictions"] > 0 and st["bytes_p2p"] > 0, st
        assert rel_err(C, Co) <= TOL
        assert np.array_equal(C, ref), n


def test_bad_scalar_tables_option():
    with pytest.raises(M.MiccoError):
        M.Context(scalar_tables=2)


needs2 = pytest.mark.skipif(torch.cuda.device_count() < 2, reason="needs >= 2 CUDA devices")


@needs2
def test_two_devices_single_process():
    """Two real devices in one process: replicas move with cudaMemcpyPeerAsync over NVLink,
    the second device's scalar table is peer-copied and accumulated on device 0."""
    wl = c5_small()
    Co = oracle.correlator(wl)
    ref, _, _ = run(wl, 1)
    for tables in (0, 1):
        C, _, st = run(wl, 2, [1, 1, 1], scalar_tables=tables, **C5_KW)
        assert st["bytes_p2p"] > 0, st
        assert np.array_equal(C, ref)
        assert rel_err(C, Co) <= TOL


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _nccl_worker(rank, world, port, q):
    """One process per GPU: identical plan on every rank, this rank's ops only, ncclSend /
    ncclRecv for cross-GPU operands, ncclAllReduce of the scalar tables."""
    import sys
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch.distributed as dist
    import paper_conf_ipps_wangr0e22_b200 as M
    from micco_inputs import workloads
    torch.cuda.set_device(rank)
    dist.init_process_group("gloo", rank=rank, world_size=world)  # plumbing only (the id)
    out = {}
    try:
        for name, wl, kw, bd in (
                ("c5_small", workloads.c5_mixed(n_combos=1, Nb=6, Nm=10, Lt=2, pool=2, meson_graphs=12),
                 dict(mem_budget_bytes=2 * 6 ** 4 * 2 * 16, window_graphs=32), [1, 1, 1]),
                ("c2_gauss", workloads.c2_meson_set(n_graphs=200, N=24, Lt=4, rate=0.7, dist="gaussian", seed=5),
                 dict(window_graphs=16), [1, 2, 0])):
            ctx = M.Context(dist_rank=rank, dist_world=world, **kw)
            M.load_workload(ctx, wl)
            obj = [M.micco_nccl_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(obj, src=0)
            M.micco_set_nccl_id(ctx.h, obj[0])
            ctx.execute(world, bd)
            C = ctx.correlator()
            st = ctx.stats()
            ctx.close()
            out[name] = (C, st["bytes_p2p"], st["evictions"])
    except Exception as e:  # reported to the parent
        out["error"] = repr(e)
    dist.destroy_process_group()
    q.put((rank, out))


@needs2
def test_two_process_nccl_world2():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_nccl_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in procs)
    for p in procs:
        p.join(timeout=120)
    refs = {"c5_small": (c5_small(), C5_KW),
            "c2_gauss": (workloads.c2_meson_set(n_graphs=200, N=24, Lt=4, rate=0.7, dist="gaussian", seed=5),
                         dict(window_graphs=16))}
    for r in (0, 1):
        assert "error" not in res[r], res[r]
    for name, (wl, kw) in refs.items():
        ref, _, _ = run(wl, 1)
        Co = oracle.correlator(wl)
        for r in (0, 1):
            C, p2p, _ = res[r][name]
            assert np.array_equal(C, ref), (name, r)  # every rank holds the all-reduced C(t)
            assert rel_err(C, Co) <= TOL
        assert res[0][name][1] > 0  # operands crossed ranks (ncclSend / ncclRecv)
