"""Host-only model of the bench's weak-scaling run (bench.py --gpus N): the plans every rank
would replay, for N = 1, 2, 4, 8, planned on the host with lazy synthetic nodes (no GPU).

Two workloads per N, both N × 10k C2 graphs (N = 128, Lt = 64, r = 0.9, Uniform):
  sets    bench.py's weak-scaling workload: N independent interleaved C2 sets
          (workloads.c2_weak_sets; set 0 is the 1-GPU workload)
  single  one C2 set of N × 10k graphs (repeats drawn from all earlier nodes)

For each, the cold plan (the e2e step: caches empty) and the warm plan (a repeat execute:
the node replicas the cold execute left cached, MICCO_PLAN_WARM=1) at the bounds the
whole-plan sweep picks, with a 163 GB budget per GPU (a B200's free memory after the
reserve).  Reported per plan: PCIe (H2D, D2H) and NVLink (P2P) bytes per GPU, evictions,
max/mean load, the modelled step time (planner cost model: per stage, max over GPUs of
flops / 30 TF/s + host bytes / 55 GB/s + peer bytes / 700 GB/s) and the modelled weak-scaling
efficiency t(1) / t(N).  A model, not a measurement: gpurun has one GPU.

Run: python tools/scale_model.py [--out profiles/scale_model_r01.json]
"""
import argparse
import json
import os
import sys
import time
from pathlib import Path

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))

import paper_conf_ipps_wangr0e22_b200 as M  # noqa: E402
from micco_inputs import workloads  # noqa: E402


def plan(wl, n, budget, warm, policy):
    ctx = M.Context(keep_inputs_resident=True, mem_budget_bytes=budget, dist_rank=0, dist_world=n, policy=policy)
    M.load_workload(ctx, wl)
    os.environ["MICCO_PLAN_WARM"] = "1" if warm else "0"
    try:
        t0 = time.perf_counter()
        st, _ = M.micco_plan(ctx.h, n, None)
        bd = list(st["reuse_bound"])
        _, _, pred = M.micco_plan_stages(ctx.h, n, "fixed", bd)
        dt = time.perf_counter() - t0
    finally:
        os.environ.pop("MICCO_PLAN_WARM", None)
        ctx.close()
    return {"n_gpus": n, "warm": warm, "policy": policy, "reuse_bound": bd, "model_s": pred,
            "h2d_gb_per_gpu": st["bytes_h2d"] / n / 1e9, "d2h_gb_per_gpu": st["bytes_d2h"] / n / 1e9,
            "p2p_gb_per_gpu": st["bytes_p2p"] / n / 1e9, "evictions": st["evictions"],
            "max_over_mean_load": st["max_over_mean_load"], "host_plan_s": dt}


def main(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--graphs", type=int, default=10000)
    ap.add_argument("--gpus", default="1,2,4,8")
    ap.add_argument("--budget-gb", type=float, default=163.0)
    ap.add_argument("--out", default=str(ROOT / "profiles" / "scale_model_r01.json"))
    a = ap.parse_args(argv)
    budget = int(a.budget_gb * 1e9)
    rows = []
    for kind, policy in (("sets", "micco_affinity"), ("sets", "micco"), ("single", "micco")):
        base = {}
        for n in [int(x) for x in a.gpus.split(",")]:
            if kind == "sets":
                wl = workloads.c2_weak_sets(n, n_graphs=a.graphs, N=128, Lt=64, rate=0.9, seed=2)
            else:
                wl = workloads.c2_meson_set(n_graphs=a.graphs * n, N=128, Lt=64, rate=0.9, seed=2)
            for warm in (False, True):
                r = plan(wl, n, budget, warm, policy)
                r["workload"] = kind
                if n == 1:
                    base[warm] = r["model_s"]
                r["model_efficiency"] = base[warm] / r["model_s"] if warm in base else None
                rows.append(r)
                print(f"{kind:6s} {policy:14s} n={n} {'warm' if warm else 'cold'}: model {r['model_s']:.3f} s "
                      f"(eff {r['model_efficiency'] or 0:.3f}), per GPU H2D {r['h2d_gb_per_gpu']:.1f} GB, "
                      f"P2P {r['p2p_gb_per_gpu']:.1f} GB, D2H {r['d2h_gb_per_gpu']:.1f} GB, "
                      f"evictions {r['evictions']}, load {r['max_over_mean_load']:.3f}", flush=True)
    meta = {"graphs_per_gpu": a.graphs, "budget_gb": a.budget_gb,
            "cost_model": "per stage max over GPUs of flops/30 TF/s + host bytes/55 GB/s + peer bytes/700 GB/s",
            "note": "host-only plans (lazy nodes); bytes, evictions and load are exact plan properties, "
                    "times are the planner's cost model, not measurements"}
    with open(a.out, "w") as f:
        json.dump({"meta": meta, "rows": rows}, f, indent=1)
    print("wrote", a.out)


if __name__ == "__main__":
    main()
