"""Bitwise reproducibility across repeated executes and fresh contexts (run on the box):
    python tools/repeat_check.py <config> [reps]
config: c3_10k | c5full | c4 | c2.  Prints the max |ΔC|/|C| between runs and whether every run
is bitwise equal to the first."""
import sys
from pathlib import Path
ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))
import numpy as np  # noqa: E402
import paper_conf_ipps_wangr0e22_b200 as M  # noqa: E402
from micco_inputs import workloads  # noqa: E402

cfg = sys.argv[1]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
budgets = [float(x) for x in sys.argv[3].split(",")] if len(sys.argv) > 3 else [0.0, 0.0]  # GB per context
if cfg == "c3_10k":
    wl, kw = workloads.c3_multi_meson(n_graphs=10000, N=256, Lt=128), dict(reorder=True)
elif cfg == "c5full":
    wl, kw = workloads.c5_mixed(n_combos=4, Nb=64, Nm=256, Lt=64, pool=4, meson_graphs=64), {}
elif cfg == "c4":
    wl, kw = workloads.c4_two_baryon(n_combos=8, N=64, Lt=64, order="greedy"), {}
else:
    wl, kw = workloads.c2_meson_set(n_graphs=10000, N=128, Lt=64, rate=0.9, seed=2), {}
out = []
for b in budgets:
    ctx = M.Context(keep_inputs_resident=True, mem_budget_bytes=int(b * 1e9), **kw)
    M.load_workload(ctx, wl)
    for r in range(reps):
        ctx.execute(1)
        C = ctx.correlator()
        vals = np.array([ctx.graph_value(g, 0) for g in range(len(wl.graphs))])
        out.append((C, vals))
        print(f"budget {b} run {r}: window {ctx.stats()['window_graphs']}", flush=True)
    ctx.close()
C0, v0 = out[0]
for i, (C, v) in enumerate(out):
    dc = np.max(np.abs(C - C0) / np.abs(C0))
    bad = np.nonzero(v != v0)[0]
    print(f"{cfg} run {i}: C bitwise {np.array_equal(C, C0)} max rel {dc:.3e}; graph values differing at t=0: {len(bad)}"
          + (f" e.g. {bad[:5].tolist()} rel {np.max(np.abs(v[bad]-v0[bad])/np.abs(v0[bad])):.2e}" if len(bad) else ""), flush=True)
    if len(bad):
        ranks = [wl.nodes[wl.graphs[g].inst[0]].rank for g in bad]
        print("   differing graphs by first-node rank:", {r: ranks.count(r) for r in set(ranks)}, flush=True)
