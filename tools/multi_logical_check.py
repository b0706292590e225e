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
