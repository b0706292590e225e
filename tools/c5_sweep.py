"""C5 memory-oversubscription sweep (§V-C, Fig. 11: memory requirement at
125% → 200% of the GPU memory; BASELINE.json configs[4]).  Run on the B200 box:

    python tools/c5_sweep.py [--out gpurun_out/c5_sweep_r02.json]

Two workloads:
  c5        the scaled C5 mixed set (bench.py --config c5: rank-4 N = 64 baryon intermediates of
            4.3 GB at Lt = 16 shared across the stream, plus N = 256 meson graphs).  Its demand =
            the plan's peak resident bytes at the fixed window W = 256 with an unbounded budget;
            budgets are set so demand / budget = 125, 150, 175, 200 %.  Each budget runs twice:
            fixed W = 256 (the paper's setting: the live set exceeds the budget, so the planner
            evicts, spills to pinned host memory and re-fetches) and the automatic window
            (options.window_graphs = 0: the largest window the budget holds without extra host
            traffic).
  c5full    C5 at its stated size (2656 graphs, N = 64 baryons, Lt = 64, 17.2 GB rank-4
            intermediates; peak resident set 153.5 GB at W = 256 with an unbounded budget): the
            same four ratios.  The automatic window runs on the GPU; the fixed W = 256 plans are
            reported host-only (not executed): they spill 0.97-1.3 TB of 17.2 GB tensors to host
            memory and re-fetch 1.7-4.5 TB per step, more than the box's 196 GB of host RAM holds
            (the first attempt was killed by the host's OOM killer).
Per run: one cold execute (nodes from pinned host memory: the e2e step) and 2 warm executes
(device-timed with CUDA events, whole call), C(t) checked bitwise equal across all runs of a
workload, graphs/s, window, evictions, H2D / D2H / P2P bytes, peak resident bytes.
"""
import argparse
import json
import os
import sys
import time
from pathlib import Path

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_wangr0e22_b200 as M  # noqa: E402
from micco_inputs import workloads  # noqa: E402


def timed(ctx):
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    ctx.execute(1)
    e.record()
    e.synchronize()
    return s.elapsed_time(e), ctx.stats()


def run(wl, budget, window, warm_steps=2):
    ctx = M.Context(keep_inputs_resident=True, mem_budget_bytes=int(budget), window_graphs=window)
    M.load_workload(ctx, wl)
    cold_ms, cst = timed(ctx)
    ms, sts = [], []
    for _ in range(warm_steps):
        m, st = timed(ctx)
        ms.append(m)
        sts.append(st)
    C = ctx.correlator()
    ctx.close()
    st = sts[-1]
    G = len(wl.graphs)
    return C, {"budget_gb": budget / 1e9, "window": st["window_graphs"], "window_mode": "fixed" if window else "auto",
               "graphs_per_s": G / (np.mean(ms) / 1e3), "ms_per_step": float(np.mean(ms)),
               "e2e_graphs_per_s": G / (cold_ms / 1e3), "e2e_ms": cold_ms,
               "evictions": st["evictions"], "bytes_h2d": st["bytes_h2d"], "bytes_d2h": st["bytes_d2h"],
               "bytes_p2p": st["bytes_p2p"], "cold_bytes_h2d": cst["bytes_h2d"], "cold_bytes_d2h": cst["bytes_d2h"],
               "peak_gb": st["peak_bytes"] / 1e9, "gemm_ms": st["gemm_kernel_ms"], "copy_ms": st["copy_ms"],
               "alloc_retries": st["alloc_retries"] + cst["alloc_retries"],
               "tflops": st["flops"] / (np.mean(ms) / 1e3) / 1e12}


def demand(wl, window):
    ctx = M.Context(mem_budget_bytes=int(10e12), window_graphs=window)
    M.load_workload(ctx, wl)
    st, _ = ctx.plan(1, [0, 0, 0])
    ctx.close()
    return st["peak_bytes"]


def main(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=str(ROOT / "gpurun_out" / "c5_sweep_r02.json"))
    ap.add_argument("--skip-full", action="store_true")
    ap.add_argument("--skip-small", action="store_true")
    a = ap.parse_args(argv)
    out = {"rows": []}
    wl = workloads.c5_mixed(n_combos=1, Nb=64, Nm=256, Lt=16, pool=2, meson_graphs=64)
    d = demand(wl, 256)
    out["c5_demand_gb"] = d / 1e9
    print(f"c5: {len(wl.graphs)} graphs, demand at W=256: {d / 1e9:.1f} GB", flush=True)
    ref = None
    for pct in ([] if a.skip_small else (125, 150, 175, 200)):
        for window in (256, 0):
            t0 = time.perf_counter()
            C, r = run(wl, d * 100 / pct, window)
            r.update({"workload": "c5", "demand_over_budget_pct": pct, "wall_s": time.perf_counter() - t0})
            ref = C if ref is None else ref
            r["bitwise_equal"] = bool(np.array_equal(C, ref))
            out["rows"].append(r)
            print(json.dumps(r), flush=True)
    if not a.skip_full:
        wl = workloads.c5_mixed(n_combos=4, Nb=64, Nm=256, Lt=64, pool=4, meson_graphs=64)
        d = demand(wl, 256)
        out["c5full_demand_gb"] = d / 1e9
        print(f"c5full: {len(wl.graphs)} graphs, demand at W=256: {d / 1e9:.1f} GB", flush=True)
        ref = None
        for pct in (125, 150, 175, 200):
            ctx = M.Context(mem_budget_bytes=int(d * 100 / pct), window_graphs=256, keep_inputs_resident=True)
            M.load_workload(ctx, wl)
            st, _ = ctx.plan(1, [0, 0, 0])
            ctx.close()
            out["rows"].append({"workload": "c5full", "demand_over_budget_pct": pct, "window": 256,
                                "window_mode": "fixed", "executed": False, "budget_gb": d / pct / 1e7,
                                "plan_bytes_h2d": st["bytes_h2d"], "plan_bytes_d2h": st["bytes_d2h"],
                                "plan_evictions": st["evictions"], "model_s": st["model_s"],
                                "model_graphs_per_s": len(wl.graphs) / st["model_s"]})
            print(json.dumps(out["rows"][-1]), flush=True)
            t0 = time.perf_counter()
            C, r = run(wl, d * 100 / pct, 0)
            r.update({"workload": "c5full", "demand_over_budget_pct": pct, "executed": True,
                      "wall_s": time.perf_counter() - t0})
            ref = C if ref is None else ref
            r["bitwise_equal"] = bool(np.array_equal(C, ref))
            out["rows"].append(r)
            print(json.dumps(r), flush=True)
    Path(a.out).parent.mkdir(parents=True, exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
