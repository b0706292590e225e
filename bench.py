#!/usr/bin/env python
"""bench.py — throughput of the MICCO hot path on B200.

One step = one micco_execute over the whole graph set: hash-consed DAG → stages → Alg. 1/2
scheduling → per-GPU HBM cache → grouped complex-FP64 DMMA GEMMs and dots → per-graph finalize
→ C(t) on the host.  Default workload: BASELINE.json configs[2], the multi-meson correlator at
its stated size (100 000 graphs, N = 256, Lt = 128; the largest single-GPU configuration), with
the reuse-aware reduction order.

    python bench.py [--gpus N --steps K --warmup W] [--impl micco|reference] [--config c3|c2|c4|c5|c5full]

* value: graphs/s with the node tensors already resident in HBM (keep_inputs_resident) when the
  timed region starts (the bench contract); inputs (8 GiB of nodes, 98 GiB of intermediates
  per step) are far larger than the 126 MB L2, so no flush is needed.
* e2e:   SURVEY.md §8(d)'s graphs/s — the same call from cold caches with the nodes in pinned
  host memory: H2D of every node used and the D2H of C(t) inside the timed region.
* roofline: the GEMM (dominant kernel), algorithmic flops ÷ its launch durations (CUDA events on
  its launching stream, inside the library), against the FP64 DMMA ceiling measured live by
  micco_probe_fp64_peak in this run (MEASURED_PEAKS.json has no FP64 entry).
  roofline_dot: the standalone dot kernel, algorithmic bytes ÷ its launch durations, against
  MEASURED_PEAKS.json hbm_gbs.
* cpu_baseline: the CPU oracle (oracle/) on a bounded sample of the same graphs, on all host
  threads and on one thread.
* secondary (N = 1): the C2 meson set (configs[1]) at repetition rate 0.9, the reuse-heavy end
  of the paper's sweep, as its own block.
Multi-GPU (torchrun, one process per GPU): c3 is strong scaling (the same 100k graphs over N
GPUs); c2 is weak scaling (N independent 10k-graph sets).  Every rank builds the identical plan,
operands move with ncclSend/ncclRecv, one ncclAllReduce combines the per-graph scalars.
policy_compare (N > 1, or --logical-gpus > 1 in one process): MICCO vs MICCO-naive vs
round-robin vs least-loaded on the repetition-heavy C2 Gaussian r = 0.9 set (§V-B).
Timing: barrier + cuda.synchronize on both sides, CUDA events, max over ranks.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

HBM_FALLBACK_GBS = 6650.0  # B200_PROFILING.md fallback (used only if MEASURED_PEAKS.json is absent)
CONFIG_GRAPHS = {"c2": 10000, "c3": 100000, "c4": 46080, "c5": 0, "c5full": 0}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="micco", choices=["micco", "reference"])
    ap.add_argument("--config", default="c3", choices=["c2", "c3", "c4", "c5", "c5full"],
                    help="c3 = BASELINE configs[2] at 100k graphs (the headline); c2 / c4 / c5 = configs[1] / [3] / [4]")
    ap.add_argument("--graphs", type=int, default=0, help="graphs (c3: total; c2: per GPU); 0 = the config's size")
    ap.add_argument("--N", type=int, default=128, help="c2 meson size")
    ap.add_argument("--Lt", type=int, default=64, help="c2 time slices")
    ap.add_argument("--rate", type=float, default=0.9, help="c2 repetition rate")
    ap.add_argument("--dist", default="uniform", choices=["uniform", "gaussian"])
    ap.add_argument("--policy", default="micco_affinity",
                    help="scheduling policy (micco_affinity = MICCO's Alg. 1/2 with the last consumer's GPU "
                         "preferred among Alg. 1's candidates; identical to micco on one GPU)")
    ap.add_argument("--window", type=int, default=0)
    ap.add_argument("--budget-gb", type=float, default=0.0,
                    help="per-GPU memory budget (0 = device free memory; c5 defaults to 25 GB: its "
                         "unconstrained plan peaks at 37.6 GB, so demand/budget = 150%%, PAPER.md L376)")
    ap.add_argument("--reorder", dest="reorder", action="store_true", default=None,
                    help="reuse-aware reduction order (options.reorder, SURVEY.md §8(f) NEXT #3); default on for c3")
    ap.add_argument("--no-reorder", dest="reorder", action="store_false")
    ap.add_argument("--logical-gpus", type=int, default=0,
                    help="single process: execute on this many logical GPUs (round-robin over the visible devices)")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--cpu-sample", type=int, default=0, help="graphs in the oracle sample (0 = auto)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-secondary", action="store_true", help="skip the C2 r = 0.9 block (N = 1)")
    ap.add_argument("--no-policy-compare", action="store_true")
    ap.add_argument("--peak-seconds", type=float, default=2.0)
    a = ap.parse_args()
    if a.reorder is None:
        a.reorder = a.config == "c3"
    if a.graphs <= 0:
        a.graphs = CONFIG_GRAPHS[a.config]
    return a


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "200"], stdout=self.f,
                                      stderr=subprocess.DEVNULL)
        except OSError:
            self.p = None
        return self

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        self.p.wait()
        self.f.flush()
        self.f.seek(0)
        rows = [r.split(",") for r in self.f.read().strip().splitlines() if r.strip()]
        sm, mx, reasons, power = [], None, set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            r = [x.strip() for x in r]
            if len(r) < 9:
                continue
            try:
                sm.append(float(r[1]))
                mx = float(r[2])
                power.append(float(r[3]))
            except ValueError:
                continue
            for nm, v in zip(names, r[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        loaded = [s for s in sm if mx and s > 0.3 * mx] or sm
        return {"sm_mhz": statistics.median(loaded) if loaded else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm),
                "power_w_max": max(power) if power else None}


def hbm_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            return float(json.load(f)["hbm_gbs"]), "of measured (MEASURED_PEAKS.json hbm_gbs)"
    except (OSError, ValueError, KeyError):
        return HBM_FALLBACK_GBS, "of fallback (B200_PROFILING.md; MEASURED_PEAKS.json absent)"


def make_workload(cfg, args, world):
    """(workload, scaling, label fields) for a config."""
    from micco_inputs import workloads
    if cfg == "c3":  # multi-meson: N = 256, Lt = 128 (configs[2]); strong scaling over GPUs
        wl = workloads.c3_multi_meson(n_graphs=args.graphs, N=256, Lt=128)
        return wl, "strong", {"N": 256, "Lt": 128, "pool": 32}
    if cfg == "c5full":  # configs[4] at its stated size: N = 64 baryons, Lt = 64, rank-4
        # intermediates of 17.2 GB, 1358 GB of intermediate demand against ~163 GB of HBM
        wl = workloads.c5_mixed(n_combos=4, Nb=64, Nm=256, Lt=64, pool=4, meson_graphs=64)
        return wl, "strong", {"Nb": 64, "Nm": 256, "Lt": 64}
    if cfg == "c5":  # oversubscribed mixed set (configs[4]) scaled to the host's RAM: rank-4
        # N = 64 intermediates of 4.3 GB (Lt = 16) shared across the stream, plus C3-style
        # N = 256 meson graphs; unconstrained peak 37.6 GB, run against a 25 GB budget
        wl = workloads.c5_mixed(n_combos=1, Nb=64, Nm=256, Lt=16, pool=2, meson_graphs=64)
        return wl, "strong", {"Nb": 64, "Nm": 256, "Lt": 16}
    if cfg == "c4":  # two-baryon: rank-3 N = 64, Lt = 64 (configs[3]); graphs = combos × 720
        wl = workloads.c4_two_baryon(n_combos=max(1, args.graphs // 720), N=64, Lt=64, order="greedy")
        return wl, "strong", {"N": 64, "Lt": 64}
    if world > 1:  # weak scaling: one independent C2 set per GPU, interleaved in one stream
        # (set 0 is the N = 1 workload); the scheduler is not told the partition
        wl = workloads.c2_weak_sets(world, n_graphs=args.graphs, N=args.N, Lt=args.Lt, rate=args.rate,
                                    dist=args.dist, seed=2)
        return wl, "weak", {"N": args.N, "Lt": args.Lt, "rate": args.rate, "dist": args.dist,
                            "graphs_per_gpu": args.graphs}
    wl = workloads.c2_meson_set(n_graphs=args.graphs, N=args.N, Lt=args.Lt, rate=args.rate, dist=args.dist, seed=2)
    return wl, "weak", {"N": args.N, "Lt": args.Lt, "rate": args.rate, "dist": args.dist}


def oracle_rate(wl, n, nthreads):
    """The oracle (as it stands) on the first n graphs: (graphs/s, seconds)."""
    import oracle
    sub = wl.subset(list(range(n)))
    table = oracle.NodeTable(sub)
    t0 = time.perf_counter()
    oracle.correlator(sub, table, nthreads=nthreads)
    dt = time.perf_counter() - t0
    return n / dt, dt


def oracle_sample_size(wl, target_s, nthreads, hint=0):
    """Graphs in a sample the oracle finishes in about target_s seconds on nthreads threads."""
    import oracle
    if hint > 0:
        return hint
    k = min(max(2, nthreads), len(wl.graphs))
    probe = wl.subset(list(range(k)))
    t0 = time.perf_counter()
    oracle.correlator(probe, nthreads=nthreads)
    dt = max(time.perf_counter() - t0, 1e-3)
    return int(max(1, min(len(wl.graphs), k * target_s / dt)))


def cpu_baseline(wl, args, target_s=12.0, one_target_s=8.0):
    nthreads = os.cpu_count() or 1
    n = oracle_sample_size(wl, target_s, nthreads, args.cpu_sample)
    rate, dt = oracle_rate(wl, n, nthreads)
    n1 = max(1, min(n, int(round(rate * one_target_s / nthreads))))
    rate1, dt1 = oracle_rate(wl, n1, 1)
    return {"value": rate, "unit": "graphs/s", "cores": nthreads, "kind": "oracle",
            "sample": f"first {n} graphs of {wl.name} ({dt:.1f} s on {nthreads} threads; naive pairwise "
                      f"contractor in complex double, no dedup, no BLAS)",
            "one_thread": {"value": rate1, "unit": "graphs/s", "cores": 1,
                           "sample": f"first {n1} graphs ({dt1:.1f} s on 1 thread)"}}


def run_block(M, torch, ctx, wl, world, n_exec, steps, warmup, e2e_steps, dist, local_rank, peak):
    """e2e (cold, inputs in pinned host memory) then warm (inputs resident) timed steps."""
    stream = torch.cuda.current_stream()

    def barrier():
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()

    def timed_execute():
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(stream)
        ctx.execute(n_exec)
        e.record(stream)
        e.synchronize()
        return s.elapsed_time(e), ctx.stats()

    def max_over_ranks(x: float) -> float:
        if dist is None:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    G = len(wl.graphs)
    e2e_ms, e2e_h2d, e2e_copy, e2e_enq, e2e_pinned = [], [], [], 0.0, 0
    ctx.release_cache()
    timed_execute()  # warm-up of the cold path (plan, allocator pools)
    for _ in range(e2e_steps):
        ctx.release_cache()
        barrier()
        ms, st = timed_execute()
        barrier()
        e2e_ms.append(max_over_ranks(ms))
        e2e_h2d.append(st["bytes_h2d"])
        e2e_copy.append(st["copy_ms"])
        e2e_enq = st["enqueue_ms"]
        e2e_pinned = st["host_pinned"]
    ctx.execute(n_exec)  # the cold run above left the nodes resident; now warm up
    for _ in range(max(3, warmup) - 1):
        ctx.execute(n_exec)
    clocks = Clocks(local_rank)
    barrier()
    clocks.start()
    step_ms, stats = [], []
    for _ in range(steps):
        ms, st = timed_execute()
        step_ms.append(ms)
        stats.append(st)
    barrier()
    clk = clocks.stop()
    total_ms = max_over_ranks(sum(step_ms))
    plan_ms_max = max_over_ranks(max(s["plan_ms"] for s in stats))
    ms_per_step = total_ms / steps
    C = ctx.correlator()

    def mean(k):
        return statistics.mean(s[k] for s in stats)

    gemm_flops = sum(s["gemm_flops"] for s in stats)
    gemm_exec = sum(s["gemm_dmma_flops"] for s in stats)
    gemm_ms = sum(s["gemm_kernel_ms"] for s in stats)
    gemm_launches = sum(s["gemm_launches"] for s in stats)
    dot_bytes = sum(s["dot_main_bytes"] for s in stats)
    dot_ms = sum(s["dot_main_ms"] for s in stats)
    achieved = gemm_flops / (gemm_ms / 1e3) / 1e12 if gemm_ms > 0 else 0.0
    executed = gemm_exec / (gemm_ms / 1e3) / 1e12 if gemm_ms > 0 else 0.0
    s0 = stats[-1]
    hbm, hbm_src = hbm_peak()
    dot_gbs = dot_bytes / (dot_ms / 1e3) / 1e9 if dot_ms > 0 else 0.0
    return {
        "value": G / (ms_per_step / 1e3), "ms_per_step": ms_per_step, "graphs": G,
        "tflops": mean("flops") / (ms_per_step / 1e3) / 1e12,
        "stats": s0, "C0": [C[0].real, C[0].imag], "clocks": clk,
        "gpu_launches": int(sum(s["kernel_launches"] for s in stats)),
        "plan_ms_max_over_ranks": plan_ms_max,
        "gemm": {"achieved": achieved, "executed": executed, "ms": gemm_ms, "launches": gemm_launches,
                 "flops_per_launch": gemm_flops / max(1, gemm_launches), "share": gemm_ms / sum(step_ms),
                 "peak": peak},
        "roofline_dot": {"bound": "hbm", "kernel": "zdot_kernel (flat / transposed dots of two tensors)",
                         "achieved": dot_gbs, "peak": hbm, "unit": "GB/s", "frac": dot_gbs / hbm,
                         "peak_source": hbm_src, "launches": int(sum(s["dot_main_launches"] for s in stats)),
                         "share_of_step": dot_ms / sum(step_ms),
                         "achieved_note": "algorithmic bytes (16 B per element of both operands, all slices) / "
                                          "dot device time (CUDA events on the launching stream, union of "
                                          "the launches' intervals)",
                         "traffic": None},
        "e2e": ({"value": G / (statistics.mean(e2e_ms) / 1e3), "unit": "graphs/s",
                 "h2d_bytes_per_step": int(statistics.mean(e2e_h2d)), "d2h_bytes_per_step": int(wl.Lt * 16),
                 "ms_per_step": statistics.mean(e2e_ms), "h2d_device_ms_per_step": statistics.mean(e2e_copy),
                 "host_enqueue_ms": e2e_enq, "host_pinned": e2e_pinned} if e2e_ms else None),
        "breakdown_ms_per_step": {"gemm": mean("gemm_kernel_ms"), "dot": mean("dot_kernel_ms"),
                                  "dot_main": mean("dot_main_ms"), "host_enqueue": mean("enqueue_ms"),
                                  "plan": mean("plan_ms")},
        "cache_per_step": {k: s0[k] for k in ("evictions", "cache_hits", "bytes_h2d", "bytes_d2h", "bytes_p2p")},
    }


def gemm_roofline(b, traffic, traffic_note):
    g = b["gemm"]
    burst, sustained = g["peak"]
    return {"bound": "tensor", "kernel": "zgemm_tma (TMA warp-specialized, meson GEMMs with M >= 128) + zgemm_persistent (cp.async, the other layouts); 3M, grouped per layout class",
            "achieved": g["achieved"], "peak": sustained, "unit": "TFLOP/s", "frac": g["achieved"] / sustained,
            "peak_source": "FP64 DMMA ceiling measured live in this run (micco_probe_fp64_peak: register-only "
                           "mma.sync m8n8k4 f64 loop, back to back, sustained); MEASURED_PEAKS.json has no FP64 entry",
            "peak_burst": burst, "traffic": traffic, "traffic_note": traffic_note,
            "gemm_launches": g["launches"], "complex_scheme": "3M (3 DMMA products per complex MAC)",
            "executed_dmma_tflops": g["executed"], "executed_frac": g["executed"] / sustained,
            "achieved_note": "algorithmic ZGEMM-convention flops (8 per complex MAC, SURVEY §8(d)) / GEMM device "
                             "time (CUDA events on the launching streams; the union of the launches' intervals, "
                             "since a chunk's launches alternate between two streams); 3M issues 3/4 of them to "
                             "the DMMA pipe",
            "gemm_share_of_step": g["share"]}


def ncu_traffic(cfg, flops_per_launch):
    """DRAM bytes per launch from a committed `ncu --set full` capture of a GEMM launch of the
    same config, scaled by flops per launch (labelled: it is not measured on this run)."""
    for name in (f"ncu_gemm_{cfg}_r02.json", f"ncu_gemm_{cfg}_r01.json"):
        p = os.path.join(ROOT, "profiles", name)
        if not os.path.exists(p):
            continue
        try:
            with open(p) as f:
                pj = json.load(f)
            t = pj["dram_bytes_per_launch"] / pj["flops_per_launch"] * flops_per_launch
            return t, (f"extrapolated: DRAM bytes per flop of one ncu --set full capture of a {cfg} GEMM launch "
                       f"(profiles/{name}) × this run's average flops per launch")
        except (OSError, ValueError, KeyError, ZeroDivisionError):
            pass
    return None, f"no ncu capture of a {cfg} GEMM launch committed"


def policy_compare(M, torch, args, world, n_exec, dist, local_rank, peak):
    """MICCO vs MICCO-naive vs round-robin vs least-loaded on the repetition-heavy C2 Gaussian
    r = 0.9 set (§V-B), one context, warm steps (inputs resident)."""
    from micco_inputs import workloads
    rank = dist.get_rank() if dist is not None else 0
    wl = workloads.c2_meson_set(n_graphs=args.graphs if args.config == "c2" else 10000, N=args.N, Lt=args.Lt,
                                rate=0.9, dist="gaussian", seed=2)
    ctx = M.Context(keep_inputs_resident=True, policy="micco", dist_rank=rank if world > 1 else 0,
                    dist_world=world if world > 1 else 0)
    if world > 1:
        obj = [M.micco_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        M.micco_set_nccl_id(ctx.h, obj[0])
    M.load_workload(ctx, wl)
    out = {"workload": f"c2_meson_set r=0.9 gaussian, {len(wl.graphs)} graphs, N={args.N}, Lt={args.Lt}",
           "n_gpus": n_exec, "steps": 3, "policies": {}}
    for pol in ("micco", "micco_affinity", "micco_naive", "round_robin", "least_loaded"):
        ctx.set_policy(pol)
        b = run_block(M, torch, ctx, wl, world, n_exec, steps=3, warmup=3, e2e_steps=1, dist=dist,
                      local_rank=local_rank, peak=peak)
        st = b["stats"]
        out["policies"][pol] = {
            "ms_per_step": b["ms_per_step"], "graphs_per_s": b["value"],
            "e2e_ms_per_step": b["e2e"]["ms_per_step"] if b["e2e"] else None,
            "bytes_h2d_cold": b["e2e"]["h2d_bytes_per_step"] if b["e2e"] else None,
            "bytes_p2p_per_step": st["bytes_p2p"], "bytes_h2d_per_step": st["bytes_h2d"],
            "cache_hits": st["cache_hits"], "max_over_mean_load": st["max_over_mean_load"],
            "sched_ms": st["sched_ms"], "sched_share": st["sched_ms"] / b["ms_per_step"],
            "reuse_bound": st["reuse_bound"]}
    rr = out["policies"]["round_robin"]["ms_per_step"]
    for v in out["policies"].values():
        v["time_vs_round_robin"] = v["ms_per_step"] / rr
    ctx.close()
    return out


def reference_arm(args, rank, world):
    """--impl reference: the CPU oracle as it stands, timed on this box's host cores, each step
    a bounded sample of the same workload (rank 0 only)."""
    if rank != 0:
        return
    import oracle
    wl, scaling, labels = make_workload(args.config, args, 1)
    nthreads = os.cpu_count() or 1
    n = oracle_sample_size(wl, 5.0, nthreads, args.cpu_sample)  # ~5 s per step: the run stays within minutes
    sub = wl.subset(list(range(n)))
    table = oracle.NodeTable(sub)
    for _ in range(args.warmup):
        oracle.correlator(sub, table, nthreads=nthreads)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.correlator(sub, table, nthreads=nthreads)
        times.append(time.perf_counter() - t0)
    ms = 1e3 * statistics.mean(times)
    value = n / (ms / 1e3)
    sample = (f"first {n} graphs of {wl.name} per step, naive pairwise contractor in complex double, "
              f"no dedup, {nthreads} threads")
    line = {
        "impl": "reference", "metric": "contraction graphs/s", "value": value, "unit": "graphs/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
        "higher_is_better": True, "scaling": scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": dict({"workload": wl.name, "graphs": len(wl.graphs), "graphs_per_step": n}, **labels),
        "cpu_baseline": {"value": value, "unit": "graphs/s", "cores": nthreads, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": "graphs/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        reference_arm(args, rank, world)
        return

    import torch
    import paper_conf_ipps_wangr0e22_b200 as M

    torch.cuda.set_device(local_rank)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", local_rank))
    n_exec = world if world > 1 else max(1, args.logical_gpus)

    # FP64 DMMA ceiling of this device, measured now (clocks sampled while it runs)
    pclk = Clocks(local_rank).start()
    peak = M.micco_probe_fp64_peak(args.peak_seconds)
    peak_clocks = pclk.stop()

    wl, scaling, labels = make_workload(args.config, args, world)
    t_setup = time.perf_counter()
    budget_gb = args.budget_gb or (25.0 if args.config == "c5" else 0.0)
    ctx = M.Context(keep_inputs_resident=True, policy=args.policy, window_graphs=args.window,
                    mem_budget_bytes=int(budget_gb * 1e9),
                    reorder=args.reorder, dist_rank=rank if world > 1 else 0, dist_world=world if world > 1 else 0)
    if world > 1:
        obj = [M.micco_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        M.micco_set_nccl_id(ctx.h, obj[0])
    M.load_workload(ctx, wl)
    t_setup = time.perf_counter() - t_setup
    b = run_block(M, torch, ctx, wl, world, n_exec, args.steps, args.warmup, args.e2e_steps, dist, local_rank, peak)
    ctx.close()

    secondary = None
    if n_exec == 1 and args.config != "c2" and not args.no_secondary:
        wl2, _, lab2 = make_workload("c2", argparse.Namespace(**dict(vars(args), graphs=10000, rate=0.9,
                                                                        dist="uniform")), 1)
        ctx2 = M.Context(keep_inputs_resident=True, policy=args.policy)
        M.load_workload(ctx2, wl2)
        b2 = run_block(M, torch, ctx2, wl2, 1, 1, steps=5, warmup=3, e2e_steps=1, dist=None,
                       local_rank=local_rank, peak=peak)
        ctx2.close()
        t2, tn2 = ncu_traffic("c2", b2["gemm"]["flops_per_launch"])
        secondary = {"workload": wl2.name, "config": dict({"graphs": len(wl2.graphs), "reduction_order": "as given"},
                                                          **lab2),
                     "value": b2["value"], "unit": "graphs/s", "ms_per_step": b2["ms_per_step"], "steps": 5,
                     "tflops": b2["tflops"], "e2e": b2["e2e"], "roofline": gemm_roofline(b2, t2, tn2),
                     "roofline_dot": b2["roofline_dot"], "clocks": b2["clocks"],
                     "breakdown_ms_per_step": b2["breakdown_ms_per_step"],
                     "unique_gemms": b2["stats"]["n_gemm"], "unique_dots": b2["stats"]["n_dot"]}

    pc = None
    if n_exec > 1 and not args.no_policy_compare:
        pc = policy_compare(M, torch, args, world, n_exec, dist, local_rank, peak)
    elif world == 1 and not args.no_policy_compare:
        # one GPU: the comparison on two logical GPUs of this device (the scheduler, cache and
        # peer-move paths run; a peer move is a device-local copy here, not NVLink)
        pc = policy_compare(M, torch, args, 1, 2, None, local_rank, peak)
        pc["note"] = ("2 logical GPUs on one B200 (micco_execute n_gpus=2 in one process): peer moves are "
                      "device-local copies, so peer-byte differences weigh less than over NVLink")

    if rank != 0:
        if dist is not None:
            dist.barrier()
            dist.destroy_process_group()
        return

    cpu = None if args.no_cpu_baseline else cpu_baseline(wl, args)
    traffic, traffic_note = ncu_traffic(args.config, b["gemm"]["flops_per_launch"])
    s0 = b["stats"]
    line = {
        "metric": "contraction graphs/s", "value": b["value"], "unit": "graphs/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": b["ms_per_step"], "higher_is_better": True,
        "scaling": scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": dict({"workload": wl.name, "graphs": b["graphs"]}, **labels, **{
            "graphs_per_gpu": labels.get("graphs_per_gpu", b["graphs"] / n_exec),
            "logical_gpus": n_exec, "policy": args.policy,
            "reduction_order": "reuse-aware (reorder)" if args.reorder else "as given",
            "budget_gb": budget_gb or None,
            "parallelism": f"task-parallel x{n_exec} (MICCO scheduler, {scaling} scaling)",
            "l2": "inputs (node tensors) and intermediates larger than L2; no flush",
            "unique_gemms": s0["n_gemm"], "unique_dots": s0["n_dot"], "dedup_hits": s0["dedup_hits"],
            "setup_s": round(t_setup, 1)}),
        "tflops": b["tflops"],
        "cache_per_step": b["cache_per_step"],
        "roofline": gemm_roofline(b, traffic, traffic_note),
        "roofline_dot": b["roofline_dot"],
        "fp64_peak_probe": {"burst_tflops": peak[0], "sustained_tflops": peak[1], "seconds": args.peak_seconds,
                            "clocks": peak_clocks},
        "cpu_baseline": cpu,
        "e2e": b["e2e"],
        "gpu_launches": b["gpu_launches"],
        "clocks": b["clocks"],
        "sched_ms_per_step": b["breakdown_ms_per_step"]["plan"],
        "plan_ms_max_over_ranks": b["plan_ms_max_over_ranks"],
        "breakdown_ms_per_step": b["breakdown_ms_per_step"],
        "correlator_t0": b["C0"],
    }
    if secondary is not None:
        line["secondary"] = secondary
    if pc is not None:
        line["policy_compare"] = pc
    print(json.dumps(line), flush=True)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
