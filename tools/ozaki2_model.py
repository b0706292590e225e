"""Numerical model of Ozaki scheme II (CRT over int8 moduli) for the complex-FP64 meson GEMM,
on the CPU with exact integer arithmetic — the accuracy half of DESIGN.md §14's estimate
(how many moduli a 1e-10 correlator needs), not a GPU implementation.

For C = A·B (N × K by K × N complex): each row of A and column of B is scaled by a power of two
so its largest |re|, |im| is just below 2^t, rounded to integers; per modulus m_i (pairwise
coprime, ≤ 256) the residues give the two K-concatenated products an int8 tensor core would form,
Tr = [Ar | Ai]·[Br ; m − Bi] and Ti = [Ar | Ai]·[Bi ; Br] (u8 × u8 → s32, exact); the Chinese
remainder theorem reconstructs the exact integer Σ_k a·b from the residues (needs Π m_i > 8·2K·2^2t),
and the scales are undone.  The error is then only the rounding of the operands to t bits.

    python tools/ozaki2_model.py [--N 256] [--seed 0]

Prints, per number of moduli, t, the max element error relative to max|C| and the error of a
tr(A·B·Y) trace (the C3 six-cycle's GEMM + fused dot), next to FP64 numpy's own errors against an
extended-precision reference.
"""
import argparse
import math

import numpy as np

MODULI = [256, 255, 253, 251, 247, 241, 239, 233, 229, 227, 223, 217, 211, 199, 197, 193, 191]


def scale_rows(X, t):
    """per-row power-of-two exponents e with max(|re|, |im|)·2^e < 2^t, and the rounded integers"""
    mx = np.maximum(np.abs(X.real), np.abs(X.imag)).max(axis=1)
    e = np.where(mx > 0, t - 1 - np.floor(np.log2(np.where(mx > 0, mx, 1.0))), 0).astype(np.int64)
    s = np.ldexp(1.0, e)[:, None]
    return e, np.rint(X.real * s).astype(np.int64), np.rint(X.imag * s).astype(np.int64)


def ozaki2_zgemm(A, B, n_mod):
    K = A.shape[1]
    mods = MODULI[:n_mod]
    M = math.prod(mods)
    t = int((math.log2(M) - math.log2(K) - 4) // 2)  # Π m_i ≥ 8·2K·2^2t
    ea, Ar, Ai = scale_rows(A, t)
    eb, BrT, BiT = scale_rows(B.T, t)  # columns of B
    Br, Bi = BrT.T, BiT.T
    Xr = np.zeros(A.shape[0] * B.shape[1], dtype=object)
    Xi = np.zeros_like(Xr)
    for m in mods:
        Mi = M // m
        w = Mi * pow(Mi, -1, m)  # CRT basis: w ≡ 1 (mod m), 0 mod the others
        ar, ai, br, bi = Ar % m, Ai % m, Br % m, Bi % m  # unsigned residues (u8 planes)
        Tr = ar @ br + ai @ ((m - bi) % m)   # [Ar | Ai]·[Br ; m − Bi]: int8 tensor-core product
        Ti = ar @ bi + ai @ br               # [Ar | Ai]·[Bi ; Br]
        assert Tr.max() < 2 ** 31 and Ti.max() < 2 ** 31
        Xr += (Tr % m).ravel().astype(object) * w
        Xi += (Ti % m).ravel().astype(object) * w

    def signed(x):
        x %= M
        return x - M if x > M // 2 else x

    Xr = np.array([signed(x) for x in Xr], dtype=object)
    Xi = np.array([signed(x) for x in Xi], dtype=object)
    sc = np.ldexp(1.0, -(ea[:, None] + eb[None, :])).ravel()
    C = np.array([float(x) for x in Xr]) * sc + 1j * (np.array([float(x) for x in Xi]) * sc)
    return C.reshape(A.shape[0], B.shape[1]), t


def ref_matmul(A, B):
    """extended-precision reference (x87 long double, 64-bit mantissa)"""
    ld = np.longdouble
    Ar, Ai, Br, Bi = (x.astype(ld) for x in (A.real, A.imag, B.real, B.imag))
    return Ar @ Br - Ai @ Bi, Ar @ Bi + Ai @ Br


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--N", type=int, default=256)
    ap.add_argument("--seed", type=int, default=0)
    a = ap.parse_args()
    rng = np.random.default_rng(a.seed)
    N = a.N

    def cplx():
        return rng.uniform(-1, 1, (N, N)) + 1j * rng.uniform(-1, 1, (N, N))

    A, B, Y = cplx(), cplx(), cplx()
    Rr, Ri = ref_matmul(A, B)
    cmax = float(np.max(np.abs(Rr.astype(float) + 1j * Ri.astype(float))))
    # trace tr(A·B·Y) = Σ_ij (AB)_ij Y_ji in long double
    ld = np.longdouble
    Yr, Yi = Y.real.astype(ld).T, Y.imag.astype(ld).T
    tr_ref = complex(float(np.sum(Rr * Yr - Ri * Yi)), float(np.sum(Rr * Yi + Ri * Yr)))

    def errs(C):
        e = float(np.max(np.abs((C.real - Rr.astype(float)) + 1j * (C.imag - Ri.astype(float)))) / cmax)
        tr = complex(np.sum(C * Y.T))
        return e, abs(tr - tr_ref) / abs(tr_ref)

    e64, t64 = errs(A @ B)
    print(f"N = K = {N}, uniform(-1, 1) complex entries, seed {a.seed}")
    print(f"FP64 numpy matmul: max |ΔC|/max|C| = {e64:.2e}, trace rel err = {t64:.2e}")
    for n_mod in (10, 11, 12, 13, 14, 15):
        C, t = ozaki2_zgemm(A, B, n_mod)
        e, te = errs(C)
        print(f"Ozaki II, {n_mod} moduli ({math.log2(math.prod(MODULI[:n_mod])):.1f} bits), t = {t}: "
              f"max |ΔC|/max|C| = {e:.2e}, trace rel err = {te:.2e}")


if __name__ == "__main__":
    main()
