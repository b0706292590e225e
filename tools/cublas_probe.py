"""Profile target: cuBLAS ZGEMM (8192^3 and batched N=128, Lt=64) so ncu can show the
library kernel's launch shape (block size, registers, smem) and DMMA-pipe activity next to
ours.  Context only; not part of the product path."""
import torch

dev = torch.device("cuda:0")
for n, lt in ((8192, 1), (128, 64)):
    a = torch.randn(lt, n, n, dtype=torch.complex128, device=dev)
    b = torch.randn(lt, n, n, dtype=torch.complex128, device=dev)
    for _ in range(3):
        c = torch.bmm(a, b)
    torch.cuda.synchronize()
