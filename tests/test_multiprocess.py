"""Multi-process (one process per GPU) host logic on CPU, world size 2, gloo.

In multi-process mode every rank adds the same nodes and graphs, builds the
identical plan, executes the tasks assigned to its GPU and exchanges operands
with matched ncclSend/ncclRecv.  Correctness therefore rests on
the plan being a pure function of the inputs: these tests run two real
processes and check, through torch.distributed (gloo), that both ranks compute
bit-identical plans and scheduler decisions, that the NCCL unique id travels
through the plumbing, and that the per-rank shares partition the task set."""
import hashlib
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import paper_conf_ipps_wangr0e22_b200 as M
    from micco_inputs import workloads
    out = {}
    wl = workloads.c2_meson_set(n_graphs=400, N=16, Lt=4, rate=0.8, dist="gaussian", seed=11)
    ctx = M.Context(mem_budget_bytes=64 * 16 * 16 * 4 * 16, window_graphs=64, dist_rank=rank, dist_world=world)
    M.load_workload(ctx, wl)
    st, _ = ctx.plan(world, [1, 2, 0])
    st, assign = M.micco_plan(ctx.h, world, [1, 2, 0], n_tasks=st["unique_tasks"])
    digest = hashlib.sha256(assign.tobytes() + repr(sorted((k, v) for k, v in st.items()
                                                             if k != "struct_size")).encode()).digest()
    # compare the plan digests across ranks
    t = torch.tensor(list(digest), dtype=torch.uint8)
    gathered = [torch.zeros_like(t) for _ in range(world)]
    dist.all_gather(gathered, t)
    out["same_plan"] = all(torch.equal(g, gathered[0]) for g in gathered)
    # this rank's share of the tasks
    mine = (assign == rank).sum()
    tot = torch.tensor([int(mine)], dtype=torch.int64)
    dist.all_reduce(tot)
    out["partition"] = int(tot.item()) == len(assign)
    out["both_used"] = bool(mine > 0)
    # NCCL id plumbing (rank 0 creates, broadcast as bytes, every rank sets it)
    try:
        uid = M.micco_nccl_unique_id() if rank == 0 else None
        obj = [uid]
        dist.broadcast_object_list(obj, src=0)
        M.micco_set_nccl_id(ctx.h, obj[0])
        out["nccl_id"] = len(obj[0]) == 128
    except M.MiccoError as e:  # NCCL not loadable on this box
        out["nccl_id"] = f"skip: {e}"
    # auto-chosen bounds agree as well
    s2, _ = ctx.plan(world, None)
    b = torch.tensor(s2["reuse_bound"], dtype=torch.int64)
    bs = [torch.zeros_like(b) for _ in range(world)]
    dist.all_gather(bs, b)
    out["same_bounds"] = all(torch.equal(x, bs[0]) for x in bs)
    ctx.close()
    dist.destroy_process_group()
    q.put((rank, out))


def test_two_ranks_build_identical_plans():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    for r in (0, 1):
        o = res[r]
        assert o["same_plan"] and o["partition"] and o["both_used"] and o["same_bounds"], o
        assert o["nccl_id"] is True or str(o["nccl_id"]).startswith("skip"), o
