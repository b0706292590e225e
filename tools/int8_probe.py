"""Probe: int8 tensor-core (IMMA via cuBLASLt, torch._int_mm) throughput on this B200,
for sizing the Ozaki-scheme FP64 emulation."""
import torch

def bench(f, iters=20):
    for _ in range(3):
        f()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(True), torch.cuda.Event(True)
    best = 1e9
    for _ in range(5):
        s.record()
        for _ in range(iters):
            f()
        e.record()
        torch.cuda.synchronize()
        best = min(best, s.elapsed_time(e) / iters)
    return best

for (m, n, k) in [(8192, 8192, 8192), (16384, 16384, 8192), (4096, 4096, 4096), (256 * 64, 128, 256), (8192, 128 * 64, 256)]:
    a = torch.randint(-127, 127, (m, k), dtype=torch.int8, device="cuda")
    b = torch.randint(-127, 127, (k, n), dtype=torch.int8, device="cuda").t().contiguous().t()
    try:
        ms = bench(lambda: torch._int_mm(a, b))
        print(f"int8 _int_mm {m}x{n}x{k}: {2*m*n*k/ms*1e-9:.1f} TOPS ({ms:.3f} ms)")
    except Exception as ex:
        print("int_mm failed", m, n, k, ex)
a = torch.randn(8192, 8192, dtype=torch.bfloat16, device="cuda")
ms = bench(lambda: a @ a)
print(f"bf16 8192^3: {2*8192**3/ms*1e-9:.1f} TFLOPS")
a8 = torch.randn(8192, 8192, device="cuda").to(torch.float8_e4m3fn)
try:
    sc = torch.tensor(1.0, device="cuda")
    ms = bench(lambda: torch._scaled_mm(a8, a8.t(), scale_a=sc, scale_b=sc, out_dtype=torch.bfloat16))
    print(f"fp8 8192^3: {2*8192**3/ms*1e-9:.1f} TFLOPS")
except Exception as ex:
    print("fp8 failed", ex)
