"""Randomized parity sweep (GPU box): random small workloads — random meson/baryon graphs at
random N (ragged sizes, both GEMM kernels, dots of every mode), meson cycles with transposes,
integer inputs — under random execution options (GPU counts 1-8 on logical GPUs, policies,
reuse bounds, windows, memory budgets that force evictions and spills, per-GPU scalar tables,
reuse-aware order, repeat executes), each checked against the CPU oracle (≤ 1e-10 relative per
time slice, bit-exact on integer inputs) and, per workload and reduction order, bitwise across
its option draws.

    python tools/fuzz_parity.py [--cases 120] [--seed 1] [--minutes 12]

Prints one line per case and a JSON summary; exits 1 on the first mismatch.
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402  (test infrastructure: the checker)
import paper_conf_ipps_wangr0e22_b200 as M  # noqa: E402
from micco_inputs import workloads  # noqa: E402
from micco_inputs.gen import GraphSpec, MODE_INT3, NodeSpec, Workload  # noqa: E402

TOL = 1e-10
POLICIES = ["micco", "micco_affinity", "micco_naive", "round_robin", "least_loaded"]


def rel_err(a, b):
    return float(np.max(np.abs(a - b) / np.maximum(np.abs(b), 1e-300)))


def draw_workload(rng, case):
    kind = rng.choice(["tiny", "mesons", "baryons"])
    mode = MODE_INT3 if rng.random() < 0.3 else 0
    Lt = int(rng.integers(1, 5))
    if kind == "tiny":
        N = int(rng.integers(2, 6))
        return workloads.tiny_random(seed=int(rng.integers(1 << 30)), n_graphs=int(rng.integers(5, 40)), N=N,
                                     Lt=Lt, mode=mode)
    if kind == "baryons":
        N = int(rng.choice([3, 4, 5, 8, 9, 16]))
        m = sorted(set(int(x) for x in rng.integers(0, 720, size=int(rng.integers(5, 60)))))
        return workloads.c4_two_baryon(n_combos=1, N=N, Lt=Lt, pool=2, order=str(rng.choice(["greedy", "chain"])),
                                       matchings=m, mode=mode)
    N = int(rng.choice([1, 5, 16, 31, 32, 33, 64, 96, 127, 128, 130, 200, 256]))
    nodes = [NodeSpec(2, N, 500 + case * 10 + i) for i in range(5)]
    graphs = []
    for _ in range(int(rng.integers(4, 30))):
        k = int(rng.integers(1, 6))
        inst = [int(x) for x in rng.integers(0, 5, size=k)]
        flips = [bool(x) for x in rng.integers(0, 2, size=k)]
        order = [int(x) for x in rng.permutation(k)]
        graphs.append(GraphSpec(inst, workloads.meson_cycle_edges(k, flips), order,
                                complex(rng.normal(), rng.normal())))
    return Workload(f"mesons{N}", Lt, case, mode, nodes, graphs)


def add_relabeled(rng, wl):
    """Append copies of random graphs with their instances relabeled (permuted), edges mapped and
    flipped end for end, and a fresh random order: the canonical component keys must match them
    to the originals (builder.cpp), and the oracle recomputes them from scratch."""
    extra = []
    for _ in range(int(rng.integers(1, 1 + len(wl.graphs)))):
        g = wl.graphs[int(rng.integers(len(wl.graphs)))]
        n = len(g.inst)
        perm = [int(x) for x in rng.permutation(n)]  # old instance u -> new index perm[u]
        inst = [0] * n
        for u in range(n):
            inst[perm[u]] = g.inst[u]
        edges = []
        for (u, p_, v, q) in g.edges:
            e = (perm[u], p_, perm[v], q)
            edges.append(e if rng.random() < 0.5 else (e[2], e[3], e[0], e[1]))
        order = [int(x) for x in rng.permutation(len(edges))]
        extra.append(GraphSpec(inst, edges, order, complex(rng.normal(), rng.normal())))
    return Workload(wl.name + "+relabeled", wl.Lt, wl.seed, wl.mode, wl.nodes, list(wl.graphs) + extra, wl.meta)


def draw_options(rng, wl):
    node_bytes = max(16 * wl.Lt * nd.N ** nd.rank for nd in wl.nodes)
    opts = {"policy": str(rng.choice(POLICIES)), "reorder": bool(rng.random() < 0.5)}
    if rng.random() < 0.4:
        opts["window_graphs"] = int(rng.integers(1, 20))
    if rng.random() < 0.3:
        opts["mem_budget_bytes"] = int(node_bytes * rng.integers(6, 20))
    if rng.random() < 0.4:
        opts["scalar_tables"] = 1
    if rng.random() < 0.3:
        opts["keep_inputs_resident"] = True
    n = int(rng.choice([1, 1, 2, 3, 4, 8]))
    bd = None if rng.random() < 0.5 else [int(x) for x in rng.integers(0, 3, size=3)]
    return opts, n, bd


def run(wl, opts, n, bd, repeats):
    ctx = M.Context(**opts)
    M.load_workload(ctx, wl)
    out = []
    for _ in range(repeats):
        ctx.execute(n, bd)
        out.append((ctx.correlator(),
                    np.array([[ctx.graph_value(g, t) for t in range(wl.Lt)] for g in range(len(wl.graphs))])))
    st = ctx.stats()
    ctx.close()
    return out, st


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cases", type=int, default=120)
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--minutes", type=float, default=12.0)
    a = ap.parse_args()
    rng = np.random.default_rng(a.seed)
    t0 = time.time()
    done, draws, evictions, p2p = 0, 0, 0, 0
    for case in range(a.cases):
        if time.time() - t0 > a.minutes * 60:
            break
        wl = draw_workload(rng, case)
        if rng.random() < 0.5:
            wl = add_relabeled(rng, wl)
        Co, valso = oracle.correlator(wl, return_values=True)
        ref = {}  # per reduction order (reorder changes the contraction trees, hence rounding)
        for _ in range(int(rng.integers(1, 4))):
            opts, n, bd = draw_options(rng, wl)
            try:
                res, st = run(wl, opts, n, bd, repeats=2 if opts.get("keep_inputs_resident") else 1)
            except M.MiccoError as e:
                if e.status == -5:  # MICCO_ERR_OOM: a drawn budget below one contraction's needs
                    continue
                raise
            draws += 1
            evictions += st["evictions"]
            p2p += st["bytes_p2p"]
            for C, vals in res:
                if wl.mode == MODE_INT3:  # graph values exact; C(t) sums random complex c_g (rounded)
                    ok = np.array_equal(vals, valso) and rel_err(C, Co) <= TOL
                else:
                    ok = rel_err(C, Co) <= TOL and all(rel_err(vals[g], valso[g]) <= TOL for g in range(len(wl.graphs)))
                if not ok:
                    errs = [rel_err(vals[g], valso[g]) for g in range(len(wl.graphs))]
                    bad = [g for g in range(len(wl.graphs)) if not (errs[g] <= TOL) or
                           (wl.mode == MODE_INT3 and not np.array_equal(vals[g], valso[g]))]
                    print(json.dumps({"FAIL": wl.name, "case": case, "mode": wl.mode, "Lt": wl.Lt, "opts": opts,
                                      "n": n, "bd": bd, "err_C": rel_err(C, Co), "bad_graphs": bad[:10],
                                      "errs": [errs[g] for g in bad[:10]],
                                      "graphs": [(wl.graphs[g].inst, wl.graphs[g].edges, wl.graphs[g].order)
                                                 for g in bad[:3]],
                                      "got": [[str(x) for x in vals[g][:2]] for g in bad[:3]],
                                      "want": [[str(x) for x in valso[g][:2]] for g in bad[:3]]}), flush=True)
                    sys.exit(1)
                key = bool(opts["reorder"])
                if key not in ref:
                    ref[key] = vals
                elif not np.array_equal(ref[key], vals):
                    print(json.dumps({"FAIL_BITWISE": wl.name, "case": case, "opts": opts, "n": n, "bd": bd}),
                          flush=True)
                    sys.exit(1)
        done += 1
        print(f"case {case}: {wl.name} graphs={len(wl.graphs)} Lt={wl.Lt} mode={wl.mode} ok", flush=True)
    print(json.dumps({"cases": done, "option_draws": draws, "evictions": int(evictions), "p2p_bytes": int(p2p),
                      "minutes": round((time.time() - t0) / 60, 1), "seed": a.seed, "result": "pass"}))


if __name__ == "__main__":
    main()
