"""Localise nondeterministic results: run a workload in fresh contexts, compare every graph value
val_g(t) with the first run bit for bit, report which (graph, slice) differ and how.
    python tools/race_hunt.py <c3_10k|c3_2k|c4|c5full> <runs> [executes_per_ctx]"""
import collections
import sys
from pathlib import Path
ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))
import numpy as np  # noqa: E402
import paper_conf_ipps_wangr0e22_b200 as M  # noqa: E402
from micco_inputs import workloads  # noqa: E402

cfg, runs = sys.argv[1], int(sys.argv[2])
per = int(sys.argv[3]) if len(sys.argv) > 3 else 1
if cfg == "c3_10k":
    wl, kw = workloads.c3_multi_meson(n_graphs=10000, N=256, Lt=128), dict(reorder=True)
elif cfg == "c3_2k":
    wl, kw = workloads.c3_multi_meson(n_graphs=2000, N=256, Lt=128), dict(reorder=True)
elif cfg == "c4":
    wl, kw = workloads.c4_two_baryon(), {}
else:
    wl, kw = workloads.c5_mixed(n_combos=4, Nb=64, Nm=256, Lt=64, pool=4, meson_graphs=64), {}
G, Lt = len(wl.graphs), wl.Lt


def ncomp(g):
    G_ = wl.graphs[g]
    parent = list(range(len(G_.inst)))

    def f(x):
        while parent[x] != x:
            x = parent[x]
        return x
    for u, _, v, _ in G_.edges:
        parent[f(u)] = f(v)
    return len({f(i) for i in range(len(G_.inst))})


ref = None
for r in range(runs):
    ctx = M.Context(keep_inputs_resident=True, **kw)
    M.load_workload(ctx, wl)
    for e in range(per):
        ctx.execute(1)
        M.micco_get_graph_value(ctx.h, 0, 0)
        vals = np.array([[ctx.graph_value(g, t) for t in range(Lt)] for g in range(G)])
        st = ctx.stats()
        if ref is None:
            ref = vals
            print(f"run {r}.{e}: reference (tma launches {st['gemm_tma_launches']}/{st['gemm_launches']})", flush=True)
            continue
        bad = np.argwhere(vals != ref)
        if len(bad) == 0:
            print(f"run {r}.{e}: bitwise equal", flush=True)
            continue
        gs = sorted(set(int(b[0]) for b in bad))
        ts = collections.Counter(int(b[1]) for b in bad)
        rel = np.abs(vals[bad[:, 0], bad[:, 1]] - ref[bad[:, 0], bad[:, 1]]) / np.abs(ref[bad[:, 0], bad[:, 1]])
        kinds = collections.Counter(ncomp(g) for g in gs)
        print(f"run {r}.{e}: {len(bad)} (g,t) differ in {len(gs)} graphs; slices {dict(ts.most_common(8))}; "
              f"components per graph {dict(kinds)}; rel diff median {np.median(rel):.2e} max {rel.max():.2e}; "
              f"graphs {gs[:12]}", flush=True)
    ctx.close()
