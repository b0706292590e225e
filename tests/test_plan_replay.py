"""Independent replay of the planner's op stream:
the executor (and, in multi-process mode, every rank) replays exactly this list, so its
invariants are the executor's correctness conditions:

* every operand of a COMPUTE is resident on that GPU (inputs uploaded, peer-copied or
  produced there earlier; a fused dot's partner too);
* a P2P copy reads a replica its source holds; an H2D reads a node or a spilled copy;
* SPILL/FREE touch only resident replicas; resident bytes never exceed the budget;
* every task of the DAG is computed exactly once (fused dots inside their GEMM).
Checked over GPU counts, policies, bounds, windows and tight budgets."""
import numpy as np
import pytest

import paper_conf_ipps_wangr0e22_b200 as M
from micco_inputs import workloads

H2D, P2P, SPILL, FREE, COMPUTE, FLUSH = range(6)


def replay(ctx, n_gpus, bd, budget):
    ops, fused = M.micco_plan_ops(ctx.h, n_gpus, bd)
    tbytes, ttask, tinfo = M.micco_dag(ctx.h)
    res = [set() for _ in range(n_gpus)]
    spilled = set()
    mem = [0] * n_gpus
    done = np.zeros(len(tinfo), dtype=np.int32)
    counts = {k: 0 for k in range(6)}
    for kind, g, src, x in ops:
        counts[kind] += 1
        if kind == H2D:
            assert x not in res[g]
            assert ttask[x] < 0 or x in spilled, "H2D of an intermediate with no host copy"
            res[g].add(x)
            mem[g] += tbytes[x]
        elif kind == P2P:
            assert src != g and x in res[src] and x not in res[g]
            res[g].add(x)
            mem[g] += tbytes[x]
        elif kind == SPILL:
            assert x in res[g] and ttask[x] >= 0
            spilled.add(x)
        elif kind == FREE:
            if g < 0:
                spilled.remove(x)
            else:
                assert x in res[g]
                res[g].remove(x)
                mem[g] -= tbytes[x]
        elif kind == COMPUTE:
            k, a, b, out = tinfo[x]
            assert a in res[g] and (b < 0 or b in res[g]), "operand not resident"
            for op in (a, b):
                if op >= 0 and ttask[op] >= 0:
                    assert done[ttask[op]] == 1, "operand produced later"
            done[x] += 1
            d = fused[x]
            if d >= 0:
                _, da, db, _ = tinfo[d]
                y = db if da == out else da
                assert y in res[g], "fused dot partner not resident"
                done[d] += 1
            elif tbytes[out] > 0:
                res[g].add(out)
                mem[g] += tbytes[out]
        if g >= 0 and kind != FLUSH:
            assert mem[g] <= budget, (kind, g, mem[g], budget)
    assert np.all(done == 1), np.nonzero(done != 1)
    return counts


@pytest.mark.parametrize("n_gpus", [1, 2, 4, 8])
@pytest.mark.parametrize("policy", ["micco", "round_robin", "least_loaded", "micco_naive"])
def test_replay_meson_set(n_gpus, policy):
    wl = workloads.c2_meson_set(n_graphs=300, N=8, Lt=2, rate=0.7, dist="gaussian", flips=True, seed=5)
    budget = 1 << 30
    ctx = M.Context(mem_budget_bytes=budget, policy=policy, window_graphs=40)
    M.load_workload(ctx, wl)
    c = replay(ctx, n_gpus, [1, 2, 0] if policy == "micco" else None, budget)
    assert c[COMPUTE] > 0 and (n_gpus == 1 or c[P2P] > 0 or policy == "round_robin")


@pytest.mark.parametrize("n_gpus", [1, 2, 3])
def test_replay_tight_budget_mixed(n_gpus):
    """C5 shape with a budget two rank-4 tensors deep: evictions and spills in the stream."""
    wl = workloads.c5_mixed(n_combos=1, Nb=6, Nm=10, Lt=2, pool=2, meson_graphs=12)
    budget = 2 * 6 ** 4 * 2 * 16
    ctx = M.Context(mem_budget_bytes=budget, window_graphs=32)
    M.load_workload(ctx, wl)
    c = replay(ctx, n_gpus, [1, 1, 1], budget)
    assert c[SPILL] > 0 and c[FREE] > 0


def test_replay_keep_inputs_and_fusion():
    wl = workloads.c2_meson_set(n_graphs=200, N=8, Lt=2, rate=0.9, seed=9)
    ctx = M.Context(mem_budget_bytes=1 << 30, keep_inputs_resident=True)
    M.load_workload(ctx, wl)
    ops, fused = M.micco_plan_ops(ctx.h, 1, [0, 0, 0])
    assert (fused >= 0).sum() > 0  # most cycles end in a fused GEMM → dot
    replay(ctx, 1, [0, 0, 0], 1 << 30)


@pytest.mark.parametrize("n_gpus", [1, 3])
def test_replay_reorder_c3(n_gpus):
    """Reuse-aware order: final dots of two level-1 products are fused into the later GEMM
    (its stage moves after the partner's producer); replay checks the partner is resident."""
    wl = workloads.c3_multi_meson(n_graphs=400, N=4, Lt=1, pool=6)
    ctx = M.Context(mem_budget_bytes=1 << 30, reorder=True, window_graphs=64)
    M.load_workload(ctx, wl)
    ops, fused = M.micco_plan_ops(ctx.h, n_gpus, [1, 1, 0])
    assert (fused >= 0).sum() > 0
    replay(ctx, n_gpus, [1, 1, 0], 1 << 30)
