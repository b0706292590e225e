"""Full-size robustness check (run on the GPU box: python tools/multi_logical_check.py) of the multi-GPU executor path on one B200: the 2-set weak-scaling
workload (2 × 10k C2 graphs, 117 GB of nodes) on 2 logical GPUs sharing the device (peer copies
become device-local copies), against 1 logical GPU: C(t) must be bitwise identical."""
import sys, time
import numpy as np
sys.path.insert(0, ".")
import paper_conf_ipps_wangr0e22_b200 as M
from micco_inputs import workloads

wl = workloads.c2_weak_sets(2, n_graphs=10000, N=128, Lt=64, rate=0.9, seed=2)
ctx = M.Context(keep_inputs_resident=True, policy="micco_affinity")
M.load_workload(ctx, wl)
res = {}
for n in (2, 1):
    ctx.release_cache()
    for rep in range(2):
        t = time.perf_counter()
        ctx.execute(n)
        dt = time.perf_counter() - t
        st = ctx.stats()
        print(f"n={n} rep={rep}: {dt*1e3:.0f} ms, p2p {st['bytes_p2p']/1e9:.1f} GB, h2d {st['bytes_h2d']/1e9:.1f} GB, "
              f"evictions {st['evictions']}, load {st['max_over_mean_load']:.3f}", flush=True)
    res[n] = ctx.correlator()
ctx.close()
print("bitwise equal n=1 vs n=2:", bool(np.array_equal(res[1], res[2])))
assert np.array_equal(res[1], res[2])


def scenario(name, wl, ns, **kw):
    """C(t) of wl on each logical GPU count in ns, one fresh context per count: bitwise equal."""
    ref = None
    for n in ns:
        c = M.Context(**kw)
        M.load_workload(c, wl)
        t = time.perf_counter()
        c.execute(n)
        dt = time.perf_counter() - t
        st = c.stats()
        C = c.correlator()
        c.close()
        print(f"{name} n={n}: {dt*1e3:.0f} ms, p2p {st['bytes_p2p']/1e9:.1f} GB, h2d {st['bytes_h2d']/1e9:.1f} GB, "
              f"d2h {st['bytes_d2h']/1e9:.1f} GB, evictions {st['evictions']}", flush=True)
        if ref is None:
            ref = C
        assert np.array_equal(C, ref), (name, n)
    print(f"{name}: bitwise equal over {ns}")


scenario("c5 25GB", workloads.c5_mixed(n_combos=1, Nb=64, Nm=256, Lt=16, pool=2, meson_graphs=64),
         (1, 2, 4), mem_budget_bytes=int(25e9), policy="micco_affinity")
scenario("c5 25GB W=256", workloads.c5_mixed(n_combos=1, Nb=64, Nm=256, Lt=16, pool=2, meson_graphs=64),
         (1, 2), mem_budget_bytes=int(25e9), window_graphs=256)
scenario("c4", workloads.c4_two_baryon(n_combos=8, N=64, Lt=64, order="greedy"), (1, 3), policy="micco_affinity")
