#!/usr/bin/env python
"""bench.py — throughput of the MICCO hot path on B200.

One step = one micco_execute over the whole C2 graph set (BASELINE.json configs[1]:
synthetic meson-only set, 10k graphs, N=128, Lt=64, repetition rate 0.9 Uniform by
default): hash-consed DAG → stages → Alg. 1/2 scheduling → per-GPU HBM cache →
grouped complex-FP64 DMMA GEMMs and dots → per-graph finalize → C(t) on the host.

    python bench.py [--gpus N --steps K --warmup W] [--impl micco|reference]

* value: graphs/s with the node tensors already resident in HBM (keep_inputs_resident;
  inputs 55 GiB ≫ the 126 MB L2, so no L2 flush is needed).
* e2e:   the same call from cold caches with the nodes in pinned host memory (H2D of every
  node used and the D2H of C(t) inside the timed region).
* roofline: the GEMM kernel (dominant), algorithmic flops ÷ its launch durations measured
  by CUDA events on its launching stream inside the library, against the measured FP64
  DMMA peak (profiles/fp64_peak_r01.txt).
* cpu_baseline: the CPU oracle (oracle/) on a bounded sample of the same graphs.
Multi-GPU (torchrun, one process per GPU): weak scaling, N independent 10k-graph C2 sets
(disjoint node pools, interleaved graph by graph; set 0 is the N = 1 workload); the plan is built
identically on every rank, operands move with ncclSend/ncclRecv, one ncclAllReduce
combines the per-graph scalars.  Timing: barrier + cuda.synchronize on both sides, CUDA
events, max over ranks.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

FP64_DMMA_PEAK_TFLOPS = 36.97   # measured, profiles/fp64_peak_r01.txt (DMMA m8n8k4 register-only)
FP64_CUBLAS_ZGEMM_TFLOPS = 36.97  # cuBLAS ZGEMM 8192^3 on the same box (profiles/fp64_peak_r01.txt)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="micco", choices=["micco", "reference"])
    ap.add_argument("--config", default="c2", choices=["c2", "c3", "c4", "c5", "c5full"],
                    help="c2 = BASELINE configs[1] (the headline); c3 / c4 = configs[2] / [3] shapes")
    ap.add_argument("--graphs", type=int, default=10000, help="graphs per GPU (weak scaling)")
    ap.add_argument("--N", type=int, default=128)
    ap.add_argument("--Lt", type=int, default=64)
    ap.add_argument("--rate", type=float, default=0.9)
    ap.add_argument("--dist", default="uniform", choices=["uniform", "gaussian"])
    ap.add_argument("--policy", default="micco_affinity",
                    help="scheduling policy (micco_affinity = MICCO's Alg. 1/2 with the last consumer's GPU "
                         "preferred among Alg. 1's candidates; identical to micco on one GPU)")
    ap.add_argument("--window", type=int, default=0)
    ap.add_argument("--budget-gb", type=float, default=0.0,
                    help="per-GPU memory budget (0 = device free memory; c5 defaults to 25 GB: its "
                         "unconstrained plan peaks at 37.6 GB, so demand/budget = 150%%, PAPER.md L376)")
    ap.add_argument("--reorder", action="store_true",
                    help="reuse-aware reduction order (options.reorder, SURVEY.md §8(f) NEXT #3)")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--cpu-sample", type=int, default=0, help="graphs in the oracle sample (0 = auto)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    return ap.parse_args()


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

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        self.p.wait()
        self.f.flush()
        self.f.seek(0)
        rows = [r.split(",") for r in self.f.read().strip().splitlines() if r.strip()]
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            r = [x.strip() for x in r]
            if len(r) < 9:
                continue
            try:
                sm.append(float(r[1]))
                mx = float(r[2])
            except ValueError:
                continue
            for nm, v in zip(names, r[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        loaded = [s for s in sm if mx and s > 0.3 * mx] or sm
        return {"sm_mhz": statistics.median(loaded) if loaded else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def c2_workload(args, world):
    from micco_inputs import workloads
    if args.config == "c3":  # multi-meson: N = 256, Lt = 128 (BASELINE configs[2])
        return workloads.c3_multi_meson(n_graphs=args.graphs * world, N=256, Lt=128)
    if args.config == "c5full":  # configs[4] at its stated size: N = 64 baryons, Lt = 64, rank-4
        # intermediates of 17.2 GB, 1358 GB of intermediate demand against ~163 GB of HBM
        return workloads.c5_mixed(n_combos=4, Nb=64, Nm=256, Lt=64, pool=4, meson_graphs=64)
    if args.config == "c5":  # oversubscribed mixed set (configs[4]), scaled to the host's RAM:
        # rank-4 N = 64 intermediates of 4.3 GB (Lt = 16) shared across the stream, plus C3-style
        # N = 256 meson graphs; unconstrained peak 37.6 GB, run against a 25 GB budget
        return workloads.c5_mixed(n_combos=1, Nb=64, Nm=256, Lt=16, pool=2, meson_graphs=64)
    if args.config == "c4":  # two-baryon: rank-3 N = 64, Lt = 64 (configs[3]); graphs = combos × 720
        return workloads.c4_two_baryon(n_combos=max(1, args.graphs * world // 720), N=64, Lt=64, order="greedy")
    if world > 1:  # weak scaling: one independent 10k-graph C2 set per GPU, interleaved in one
        # stream (set 0 is the N = 1 workload); the scheduler is not told the partition
        return workloads.c2_weak_sets(world, n_graphs=args.graphs, N=args.N, Lt=args.Lt, rate=args.rate,
                                      dist=args.dist, seed=2)
    return workloads.c2_meson_set(n_graphs=args.graphs, N=args.N, Lt=args.Lt, rate=args.rate,
                                  dist=args.dist, seed=2)


def oracle_sample_rate(wl, n_graphs_hint: int):
    """Time the oracle (as it stands) on the first graphs of the workload; returns
    (graphs/s, graphs, seconds, threads)."""
    import oracle
    nthreads = os.cpu_count() or 1
    n = n_graphs_hint
    if n <= 0:  # auto: probe with a few graphs, then size the sample for ~15 s
        probe = wl.subset(list(range(min(8, len(wl.graphs)))))
        t0 = time.perf_counter()
        oracle.correlator(probe, nthreads=nthreads)
        dt = max(time.perf_counter() - t0, 1e-3)
        n = int(max(8, min(len(wl.graphs), len(probe.graphs) * 15.0 / dt)))
    sub = wl.subset(list(range(n)))
    table = oracle.NodeTable(sub)
    t0 = time.perf_counter()
    oracle.correlator(sub, table, nthreads=nthreads)
    dt = time.perf_counter() - t0
    return n / dt, n, dt, nthreads


def reference_arm(args, rank, world):
    """--impl reference: the CPU oracle as it stands, timed on this box's host cores,
    each step a bounded sample of the same workload (rank 0 only)."""
    if rank != 0:
        return
    import oracle
    wl = c2_workload(args, 1)
    nthreads = os.cpu_count() or 1
    rate, n, dt, _ = oracle_sample_rate(wl, args.cpu_sample if args.cpu_sample else 0)
    n = max(8, int(n * 6.0 / 15.0))  # keep the whole --steps/--warmup run within minutes
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
    sample = f"first {n} graphs of {wl.name} (N={args.N}, Lt={args.Lt}), naive pairwise contractor, no dedup"
    line = {
        "impl": "reference", "metric": "contraction graphs/s", "value": value, "unit": "graphs/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": wl.name, "graphs_per_step": n, "N": args.N, "Lt": args.Lt, "rate": args.rate,
                   "dist": args.dist},
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

    def barrier():
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()

    wl = c2_workload(args, world)
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
    G = len(wl.graphs)
    stream = torch.cuda.current_stream()

    def timed_execute():
        """One step bracketed by CUDA events on this process's stream (the library call is
        synchronous, so the stop event is recorded after all its device work)."""
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(stream)
        ctx.execute(world)
        e.record(stream)
        e.synchronize()
        return s.elapsed_time(e), ctx.stats()

    def max_over_ranks(x: float) -> float:
        if dist is None:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    # ---- e2e: cold caches, node tensors in pinned host memory
    e2e_ms, e2e_h2d, e2e_d2h, e2e_copy = [], [], [], []
    ctx.release_cache()
    timed_execute()  # warm-up of the cold path (plan, allocator pools)
    for _ in range(args.e2e_steps):
        ctx.release_cache()
        barrier()
        ms, st = timed_execute()
        barrier()
        e2e_ms.append(max_over_ranks(ms))
        e2e_h2d.append(st["bytes_h2d"])
        e2e_copy.append(st["copy_ms"])
        e2e_enq = st["enqueue_ms"]
        e2e_pinned = st["host_pinned"]
        e2e_d2h.append(wl.Lt * 16)
    # ---- warm: inputs resident in HBM (left cached by the cold run)
    ctx.execute(world)
    for _ in range(max(3, args.warmup) - 1):
        ctx.execute(world)
    clocks = Clocks(local_rank)
    barrier()
    clocks.start()
    step_ms, stats = [], []
    for _ in range(args.steps):
        ms, st = timed_execute()
        step_ms.append(ms)
        stats.append(st)
    barrier()
    clk = clocks.stop()
    total_ms = max_over_ranks(sum(step_ms))
    ms_per_step = total_ms / args.steps
    value = G / (ms_per_step / 1e3)
    C = ctx.correlator()

    gemm_flops = sum(s["gemm_flops"] for s in stats)
    gemm_exec_flops = sum(s["gemm_dmma_flops"] for s in stats)
    gemm_ms = sum(s["gemm_kernel_ms"] for s in stats)
    gemm_launches = sum(s["gemm_launches"] for s in stats)
    achieved = gemm_flops / (gemm_ms / 1e3) / 1e12 if gemm_ms > 0 else 0.0
    executed = gemm_exec_flops / (gemm_ms / 1e3) / 1e12 if gemm_ms > 0 else 0.0
    flops_step = statistics.mean(s["flops"] for s in stats)
    launches = int(sum(s["kernel_launches"] for s in stats))

    if rank != 0:
        if dist is not None:
            dist.barrier()
            dist.destroy_process_group()
        return

    cpu = None
    if not args.no_cpu_baseline:
        rate, n, dt, nthreads = oracle_sample_rate(wl, args.cpu_sample)
        cpu = {"value": rate, "unit": "graphs/s", "cores": nthreads, "kind": "oracle",
               "sample": f"first {n} graphs of {wl.name} ({dt:.1f} s on {nthreads} threads; naive pairwise "
                         f"contractor, no dedup, no BLAS)"}
    traffic = None
    prof = os.path.join(ROOT, "profiles", "ncu_gemm_r01.json")
    if os.path.exists(prof):
        try:
            with open(prof) as f:
                pj = json.load(f)
            if pj.get("flops_per_launch"):
                # scale the profiled DRAM bytes per flop to this run's average launch
                traffic = pj["dram_bytes_per_launch"] / pj["flops_per_launch"] * (gemm_flops / max(1, gemm_launches))
        except (OSError, ValueError, KeyError):
            traffic = None
    s0 = stats[-1]
    line = {
        "metric": "contraction graphs/s", "value": value, "unit": "graphs/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": wl.name, "graphs": G, "graphs_per_gpu": args.graphs,
                   "N": wl.meta.get("N", args.N), "Lt": wl.Lt,
                   "rate": args.rate if args.config == "c2" else None,
                   "dist": args.dist if args.config == "c2" else None, "policy": args.policy,
                   "reduction_order": "reuse-aware (reorder)" if args.reorder else "as given",
                   "budget_gb": budget_gb or None,
                   "parallelism": f"task-parallel x{world} (MICCO scheduler)",
                   "l2": "inputs (node tensors) larger than L2; no flush",
                   "unique_gemms": s0["n_gemm"], "unique_dots": s0["n_dot"], "dedup_hits": s0["dedup_hits"],
                   "setup_s": round(t_setup, 1)},
        "tflops": flops_step / (ms_per_step / 1e3) / 1e12,
        "cache_per_step": {k: s0[k] for k in ("evictions", "cache_hits", "bytes_h2d", "bytes_d2h", "bytes_p2p")},
        "roofline": {"bound": "tensor", "kernel": "zgemm_persistent (3M, grouped per layout class)", "achieved": achieved,
                     "peak": FP64_DMMA_PEAK_TFLOPS, "unit": "TFLOP/s", "frac": achieved / FP64_DMMA_PEAK_TFLOPS,
                     "peak_source": "measured FP64 DMMA microbenchmark (profiles/fp64_peak_r01.txt); "
                                    "MEASURED_PEAKS.json has no FP64 entry",
                     "traffic": traffic, "gemm_launches": gemm_launches,
                     "complex_scheme": "3M (3 DMMA products per complex MAC)" if stats[-1]["gemm_3m"] else "4M",
                     "executed_dmma_tflops": executed, "executed_frac": executed / FP64_DMMA_PEAK_TFLOPS,
                     "achieved_note": "algorithmic ZGEMM-convention flops (8 per complex MAC, SURVEY §8(d)) / "
                                      "GEMM launch time (CUDA events on the launching stream)",
                     "gemm_share_of_step": gemm_ms / sum(step_ms)},
        "cpu_baseline": cpu,
        "e2e": ({"value": G / (statistics.mean(e2e_ms) / 1e3), "unit": "graphs/s",
                 "h2d_bytes_per_step": int(statistics.mean(e2e_h2d)), "d2h_bytes_per_step": int(e2e_d2h[0]),
                 "ms_per_step": statistics.mean(e2e_ms),
                 "h2d_device_ms_per_step": statistics.mean(e2e_copy),
                 "host_enqueue_ms": e2e_enq, "host_pinned": e2e_pinned} if e2e_ms else None),
        "gpu_launches": launches,
        "clocks": clk,
        "sched_ms_per_step": statistics.mean(s["sched_ms"] for s in stats),
        "breakdown_ms_per_step": {"gemm": statistics.mean(s["gemm_kernel_ms"] for s in stats),
                                  "dot": statistics.mean(s["dot_kernel_ms"] for s in stats),
                                  "host_enqueue": statistics.mean(s["enqueue_ms"] for s in stats)},
        "correlator_t0": [C[0].real, C[0].imag],
    }
    print(json.dumps(line), flush=True)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
