"""Scheduler comparison on the reuse-vs-balance sets (SURVEY.md §8(d) "Scheduler comparison";
PAPER.md L305-360, the repetition-rate / distribution sweep of §5).

For C2-shaped meson sets (k ∈ {3, 4} cycles, N = 128, Lt = 64) over repetition rate r and
Uniform / Gaussian node selection, at 2 / 4 / 8 GPUs, every policy is planned on the host
(no GPU, no tensor data: lazy synthetic nodes) with the per-GPU budget of a B200 (180 GB):

  micco         Alg. 1 + Alg. 2 with reuse bounds from the whole-plan sweep
  micco_naive   Alg. 2 only (no reuse classification)
  round_robin   pair i of a vector on GPU i mod n
  least_loaded  Groute's rule: the GPU with the least assigned work

and reports per plan: the modelled time (planner cost model: per stage, max over GPUs of
flops / 42.9 TF/s + host bytes / 55.5 GB/s + peer bytes / 770 GB/s), H2D and P2P bytes, cache
hits, evictions, max/mean load and the host planning time (host_s).  The modelled time is a model,
not a measurement (the GPU box has one B200); bytes, hits and load balance are exact
properties of the plans the executor replays.

Run: python tools/policy_study.py [--graphs 10000] [--out profiles/policy_study_r01.json]
"""
import argparse
import json
import sys
import time
from pathlib import Path

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))

import paper_conf_ipps_wangr0e22_b200 as M  # noqa: E402
from micco_inputs import workloads  # noqa: E402

POLICIES = ["micco", "micco_affinity", "micco_naive", "round_robin", "least_loaded"]


def plan(wl, policy, n_gpus, window, budget):
    ctx = M.Context(mem_budget_bytes=budget, window_graphs=window, dist_world=1, policy=policy)
    M.load_workload(ctx, wl)
    t0 = time.perf_counter()
    _, _, pred = M.micco_plan_stages(ctx.h, n_gpus, "fixed", None)
    st, _ = M.micco_plan(ctx.h, n_gpus, None)
    dt = time.perf_counter() - t0
    ctx.close()
    return {"policy": policy, "n_gpus": n_gpus, "model_s": pred, "bytes_h2d": st["bytes_h2d"],
            "bytes_p2p": st["bytes_p2p"], "cache_hits": st["cache_hits"], "evictions": st["evictions"],
            "max_over_mean_load": st["max_over_mean_load"],
            "reuse_bound": list(st["reuse_bound"]), "unique_gemms": st["n_gemm"], "host_s": dt}


def main(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--graphs", type=int, default=10000)
    ap.add_argument("--N", type=int, default=128)
    ap.add_argument("--Lt", type=int, default=64)
    ap.add_argument("--window", type=int, default=64)
    ap.add_argument("--budget-gb", type=float, default=180.0)
    ap.add_argument("--rates", default="0.1,0.3,0.5,0.7,0.9")
    ap.add_argument("--gpus", default="2,4,8")
    ap.add_argument("--out", default=str(ROOT / "profiles" / "policy_study_r01.json"))
    a = ap.parse_args(argv)
    rows = []
    for dist in ("uniform", "gaussian"):
        for r in [float(x) for x in a.rates.split(",")]:
            wl = workloads.c2_meson_set(n_graphs=a.graphs, N=a.N, Lt=a.Lt, rate=r, dist=dist, seed=2)
            for n in [int(x) for x in a.gpus.split(",")]:
                base = None
                for pol in POLICIES:
                    res = plan(wl, pol, n, a.window, int(a.budget_gb * 1e9))
                    res.update(dist=dist, rate=r)
                    if pol == "round_robin":
                        base = res
                    rows.append(res)
                for res in rows[-len(POLICIES):]:
                    res["model_vs_round_robin"] = res["model_s"] / base["model_s"]
                line = "  ".join(f"{x['policy']}={x['model_s']:.3f}s/{x['bytes_h2d'] / 1e9:.0f}GB"
                                 for x in rows[-len(POLICIES):])
                print(f"{dist:8s} r={r:.1f} n={n}: {line}", flush=True)
    meta = {"graphs": a.graphs, "N": a.N, "Lt": a.Lt, "window_graphs": a.window, "budget_gb": a.budget_gb,
            "cost_model": "per stage max over GPUs of flops/42.9 TF/s + host bytes/55.5 GB/s + peer bytes/770 GB/s",
            "note": "modelled plan time (host-only planning); bytes, hits and load are exact plan properties"}
    Path(a.out).write_text(json.dumps({"meta": meta, "rows": rows}, indent=1))
    print("wrote", a.out)


if __name__ == "__main__":
    main()
