"""Host-only model of bench.py's multi-GPU runs (--gpus N): the plans every rank would replay,
for N = 1, 2, 4, 8, planned on the host with lazy synthetic nodes (no GPU).

Workloads:
  c3      the default bench config, strong scaling: the same 100k C3 graphs (N = 256, Lt = 128,
          reuse-aware order) on N GPUs
  sets    bench.py --config c2, weak scaling: N independent interleaved 10k-graph C2 sets
          (workloads.c2_weak_sets; set 0 is the 1-GPU workload; N = 128, Lt = 64, r = 0.9)
  single  one C2 set of N × 10k graphs (repeats drawn from all earlier nodes)

For each, the cold plan (the e2e step: caches empty) and the warm plan (a repeat execute:
the node replicas the cold execute left cached, MICCO_PLAN_WARM=1) at the bounds the
whole-plan sweep picks, with a 163 GB budget per GPU (a B200's free memory after the
reserve).  Reported per plan: PCIe (H2D, D2H) and NVLink (P2P) bytes per GPU, evictions,
max/mean load, the modelled GPU time of a step (planner cost model, core.h kModel*: per stage,
max over GPUs of flops / 42.9 TF/s + host bytes / 55.5 GB/s + peer bytes / 770 GB/s), the
host time of one plan (every rank plans the whole DAG once per execute, on a thread that
streams stages to the executor), and two step models: `overlapped` = max(GPU, plan) (planning
streams ahead of the replay, and each GPU's H2D and peer copies overlap its kernels on their
own streams: per stage max(flops, host, peer) time) and `serial` = GPU + plan (copies
serialised with the kernels, no planning overlap: the pessimistic bound).
Efficiency: strong scaling t(1) / (N · t(N)); weak scaling t(1) / t(N).  A model, not a
measurement: gpurun has one GPU.

Run: python tools/scale_model.py [--out profiles/r02/scale_model_r02.json] [--kinds c3,sets]
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


def plan(wl, n, budget, warm, policy, reorder=False, cold_plan_s=0.0):
    """(warm: the host API plans a cold execute first, then the repeat from its final
    residency; cold_plan_s, the cold plan's time measured just before, is subtracted.)"""
    ctx = M.Context(keep_inputs_resident=True, mem_budget_bytes=budget, dist_rank=0, dist_world=n, policy=policy,
                    reorder=reorder)
    M.load_workload(ctx, wl)
    os.environ["MICCO_PLAN_WARM"] = "1" if warm else "0"
    try:
        t0 = time.perf_counter()
        st, _ = M.micco_plan(ctx.h, n, None)  # the first execute's bound sweep (27 plans)
        sweep_s = time.perf_counter() - t0
        bd = list(st["reuse_bound"])
        t0 = time.perf_counter()
        st, _ = M.micco_plan(ctx.h, n, bd)    # what every later execute plans (one plan)
        plan_s = time.perf_counter() - t0 - (cold_plan_s if warm else 0.0)
        _, _, pred = M.micco_plan_stages(ctx.h, n, "fixed", bd)
    finally:
        os.environ.pop("MICCO_PLAN_WARM", None)
        ctx.close()
    ov = st["model_overlap_s"]
    return {"n_gpus": n, "warm": warm, "policy": policy, "reuse_bound": bd, "model_gpu_s": pred,
            "model_gpu_copies_overlapped_s": ov, "host_plan_s": plan_s, "host_sweep_s": sweep_s,
            "model_step_overlapped_s": max(ov, plan_s), "model_step_serial_s": pred + plan_s,
            "h2d_gb_per_gpu": st["bytes_h2d"] / n / 1e9, "d2h_gb_per_gpu": st["bytes_d2h"] / n / 1e9,
            "p2p_gb_per_gpu": st["bytes_p2p"] / n / 1e9, "evictions": st["evictions"],
            "max_over_mean_load": st["max_over_mean_load"]}


def main(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--graphs", type=int, default=10000, help="C2 graphs per GPU")
    ap.add_argument("--c3-graphs", type=int, default=100000)
    ap.add_argument("--gpus", default="1,2,4,8")
    ap.add_argument("--kinds", default="c3,sets,single")
    ap.add_argument("--budget-gb", type=float, default=163.0)
    ap.add_argument("--out", default=str(ROOT / "profiles" / "r02" / "scale_model_r02.json"))
    a = ap.parse_args(argv)
    budget = int(a.budget_gb * 1e9)
    rows = []
    kinds = a.kinds.split(",")
    cases = [(k, p) for k, p in (("c3", "micco_affinity"), ("sets", "micco_affinity"), ("sets", "micco"),
                                 ("single", "micco")) if k in kinds]
    for kind, policy in cases:
        base = {}
        strong = kind == "c3"
        for n in [int(x) for x in a.gpus.split(",")]:
            if kind == "c3":
                wl = workloads.c3_multi_meson(n_graphs=a.c3_graphs, N=256, Lt=128)
            elif kind == "sets":
                wl = workloads.c2_weak_sets(n, n_graphs=a.graphs, N=128, Lt=64, rate=0.9, seed=2)
            else:
                wl = workloads.c2_meson_set(n_graphs=a.graphs * n, N=128, Lt=64, rate=0.9, seed=2)
            cold_s = 0.0
            for warm in (False, True):
                r = plan(wl, n, budget, warm, policy, reorder=strong, cold_plan_s=cold_s)
                cold_s = r["host_plan_s"]
                r["workload"] = kind
                r["scaling"] = "strong" if strong else "weak"
                for key in ("model_gpu_s", "model_gpu_copies_overlapped_s", "model_step_overlapped_s", "model_step_serial_s"):
                    if n == 1:
                        base[(warm, key)] = r[key]
                    b = base.get((warm, key))
                    eff = None if b is None else (b / (n * r[key]) if strong else b / r[key])
                    r["eff_" + key[len("model_"):-len("_s")]] = eff
                rows.append(r)
                print(f"{kind:6s} {policy:14s} n={n} {'warm' if warm else 'cold'}: GPU {r['model_gpu_s']:.3f} s, "
                      f"plan {r['host_plan_s']:.3f} s (sweep {r['host_sweep_s']:.2f} s) -> eff overlapped "
                      f"{r['eff_step_overlapped'] or 0:.3f} serial {r['eff_step_serial'] or 0:.3f}; per GPU "
                      f"H2D {r['h2d_gb_per_gpu']:.1f} GB, P2P {r['p2p_gb_per_gpu']:.1f} GB, "
                      f"D2H {r['d2h_gb_per_gpu']:.1f} GB, evictions {r['evictions']}, "
                      f"load {r['max_over_mean_load']:.3f}", flush=True)
    meta = {"c2_graphs_per_gpu": a.graphs, "c3_graphs": a.c3_graphs, "budget_gb": a.budget_gb,
            "cost_model": "per stage max over GPUs of flops/42.9 TF/s + host bytes/55.5 GB/s + peer bytes/770 GB/s",
            "host": f"{os.cpu_count()} threads of the build container",
            "note": "host-only plans (lazy nodes); bytes, evictions and load are exact plan properties, "
                    "GPU times are the planner's cost model, plan times are measured on this host"}
    Path(a.out).parent.mkdir(parents=True, exist_ok=True)
    with open(a.out, "w") as f:
        json.dump({"meta": meta, "rows": rows}, f, indent=1)
    print("wrote", a.out)


if __name__ == "__main__":
    main()
