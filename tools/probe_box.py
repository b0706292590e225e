"""One-off probe of the GPU box: host cores/RAM, H2D/D2H pinned bandwidth, and
cuBLAS DGEMM / ZGEMM throughput (the library FP64 ceiling next to the DMMA
microbenchmark in tools/fp64_peak.cu).  Output is summarised in
profiles/fp64_peak_r01.txt.  Not part of the product path."""
import os
import subprocess
import time

import torch


def timed(fn, reps=5):
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    fn()
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(reps):
        s.record()
        fn()
        e.record()
        e.synchronize()
        best = min(best, s.elapsed_time(e))
    return best


def main():
    print("nproc", os.cpu_count(), "sched_getaffinity", len(os.sched_getaffinity(0)))
    print(subprocess.run(["free", "-g"], capture_output=True, text=True).stdout)
    print(subprocess.run(["nvidia-smi", "--query-gpu=name,memory.total,clocks.sm,clocks.max.sm,power.limit",
                          "--format=csv"], capture_output=True, text=True).stdout)
    dev = torch.device("cuda:0")
    nbytes = 1 << 30
    h = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    d = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    ms = timed(lambda: d.copy_(h, non_blocking=True))
    print(f"H2D pinned 1 GiB: {nbytes / ms * 1e-6:.1f} GB/s")
    ms = timed(lambda: h.copy_(d, non_blocking=True))
    print(f"D2H pinned 1 GiB: {nbytes / ms * 1e-6:.1f} GB/s")
    t0 = time.time()
    big = torch.empty(8 << 30, dtype=torch.uint8).pin_memory()
    print(f"pin 8 GiB host alloc: {time.time() - t0:.2f} s")
    del big
    for n in (4096, 8192):
        a = torch.randn(n, n, dtype=torch.float64, device=dev)
        b = torch.randn(n, n, dtype=torch.float64, device=dev)
        ms = timed(lambda: a @ b)
        print(f"cuBLAS DGEMM {n}^3: {2 * n**3 / ms * 1e-9:.2f} TFLOP/s ({ms:.2f} ms)")
        ac = torch.complex(a, b)
        bc = torch.complex(b, a)
        ms = timed(lambda: ac @ bc)
        print(f"cuBLAS ZGEMM {n}^3: {8 * n**3 / ms * 1e-9:.2f} TFLOP/s ({ms:.2f} ms)")
    # batched ZGEMM at the meson shapes (cfg2 N=128 Lt=64, cfg3 N=256 Lt=128)
    for n, lt in ((128, 64), (256, 128)):
        a = torch.randn(lt, n, n, dtype=torch.complex128, device=dev)
        b = torch.randn(lt, n, n, dtype=torch.complex128, device=dev)
        ms = timed(lambda: torch.bmm(a, b))
        print(f"cuBLAS batched ZGEMM N={n} Lt={lt}: {8 * n**3 * lt / ms * 1e-9:.2f} TFLOP/s ({ms * 1e3:.1f} us)")


if __name__ == "__main__":
    main()
