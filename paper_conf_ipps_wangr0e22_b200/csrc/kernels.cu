// kernels.cu — the contraction kernels of the hot path, hand-written for sm_100a.
//
// FP64 on B200 has no tcgen05/UMMA kind (ptxas rejects .kind::f64; SURVEY.md §0 probe 2):
// the FP64 tensor instruction is the warp-level DMMA.8x8x4 (mma.sync m8n8k4 f64), which
// shares one issue pipe with DFMA.  Measured ceiling on the box: 36.97 TFLOP/s
// (profiles/fp64_peak_r01.txt).  The GEMM below keeps that pipe fed from a 4-stage
// cp.async shared-memory pipeline, with 32×32-complex warp tiles (64 independent DMMAs per
// k-quad per warp, 128 FP64 accumulator registers per thread).
//
// Complex arithmetic on the real DMMA: per 8×8×4 complex block,
//   Cr += Ar·Br + (−Ai)·Bi,   Ci += Ar·Bi + Ai·Br          (4 DMMAs, 8 real flops / complex MAC)
// with −Ai formed by flipping the sign bit (integer ALU, not the FP64 pipe).  No conjugation
// anywhere (SURVEY.md §8(c) reading #7).
#include <cstdio>
#include <cstdlib>

#include "kernels.h"

namespace micco {
namespace {

constexpr int BM = kGemmBM, BN = kGemmBN, BK = kGemmBK, ST = kGemmStages, NT = kGemmThreads;
constexpr int APITCH = BK + 4;  // complex per A row: 192 B → fragment loads conflict-free
constexpr int BPITCH = BN + 2;  // complex per B row: 1056 B ≡ 32 (mod 128) → conflict-free
constexpr int A_STAGE = BM * APITCH;
constexpr int B_STAGE = BK * BPITCH;
constexpr int GEMM_SMEM = ST * (A_STAGE + B_STAGE) * 16;

__device__ __forceinline__ void cp_async16(void *smem, const void *gmem, bool valid) {
  unsigned s = (unsigned)__cvta_generic_to_shared(smem);
  int sz = valid ? 16 : 0;  // src-size 0 → zero fill (ragged tiles)
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(s), "l"(gmem), "r"(sz));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;\n" ::"n"(N));
}

// D(8x8) += A(8x4, row) · B(4x8, col), FP64 tensor core.
// Fragments: a = A[lane/4][lane%4], b = B[lane%4][lane/4], d = D[lane/4][2*(lane%4) + {0,1}].
__device__ __forceinline__ void dmma(double &d0, double &d1, double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
      : "+d"(d0), "+d"(d1)
      : "d"(a), "d"(b));
}

__device__ __forceinline__ double dneg(double x) {
  return __longlong_as_double(__double_as_longlong(x) ^ (long long)0x8000000000000000ULL);
}

template <typename D>
__device__ __forceinline__ int find_desc(const D *descs, int n, long long item) {
  int lo = 0, hi = n - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (descs[mid].tile_begin <= item) lo = mid; else hi = mid - 1;
  }
  return lo;
}

__device__ __forceinline__ void zgemm_dmma_kernel_body(const GemmDesc *__restrict__ descs, int n_desc,
                                                       long long total) {
  extern __shared__ __align__(128) double2 smem[];
  double2 *As = smem;
  double2 *Bs = smem + ST * A_STAGE;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int wm = warp >> 1, wn = warp & 1;

  for (long long tile = blockIdx.x; tile < total; tile += gridDim.x) {
    const GemmDesc &d = descs[find_desc(descs, n_desc, tile)];
    long long lt = tile - d.tile_begin;
    const int tn = (int)(lt % d.tilesN); lt /= d.tilesN;
    const int tm = (int)(lt % d.tilesM); lt /= d.tilesM;
    const int no = (int)(lt % d.No); lt /= d.No;
    const int mo = (int)(lt % d.Mo);
    const int t = (int)(lt / d.Mo);
    const int m0 = tm * BM, n0 = tn * BN;
    const int Mi = d.Mi, Ni = d.Ni, Ki = d.Ki;
    const long long sAmi = d.sAmi, sAki = d.sAki, sBki = d.sBki, sBni = d.sBni;
    const long long sAko = d.sAko, sBko = d.sBko;
    const double2 *Abase = d.A + t * d.sAt + mo * d.sAmo + m0 * sAmi;
    const double2 *Bbase = d.B + t * d.sBt + no * d.sBno + n0 * sBni;
    const bool a_kfast = (sAki == 1);   // A row-major over (m, k): copy along k
    const bool b_nfast = (sBni == 1);   // B row-major over (k, n): copy along n
    const int KT = (Ki + BK - 1) / BK;
    const int KTOT = d.Ko * KT;

    auto load_stage = [&](int slot, int kt) {
      const int ko = kt / KT;
      const int kb = (kt - ko * KT) * BK;
      const double2 *Ak = Abase + ko * sAko;
      const double2 *Bk = Bbase + ko * sBko;
      double2 *as = As + slot * A_STAGE;
      double2 *bs = Bs + slot * B_STAGE;
#pragma unroll
      for (int j = 0; j < (BM * BK) / NT; ++j) {
        const int e = tid + j * NT;
        int m, k;
        if (a_kfast) { k = e & (BK - 1); m = e / BK; } else { m = e & (BM - 1); k = e / BM; }
        const bool v = (m0 + m < Mi) && (kb + k < Ki);
        const double2 *src = v ? Ak + (long long)m * sAmi + (long long)(kb + k) * sAki : d.A;
        cp_async16(as + m * APITCH + k, src, v);
      }
#pragma unroll
      for (int j = 0; j < (BN * BK) / NT; ++j) {
        const int e = tid + j * NT;
        int n, k;
        if (b_nfast) { n = e & (BN - 1); k = e / BN; } else { k = e & (BK - 1); n = e / BK; }
        const bool v = (n0 + n < Ni) && (kb + k < Ki);
        const double2 *src = v ? Bk + (long long)(kb + k) * sBki + (long long)n * sBni : d.B;
        cp_async16(bs + k * BPITCH + n, src, v);
      }
    };

    double cr[4][4][2], ci[4][4][2];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) { cr[i][j][0] = cr[i][j][1] = ci[i][j][0] = ci[i][j][1] = 0.0; }

#pragma unroll
    for (int s = 0; s < ST - 1; ++s) {
      if (s < KTOT) load_stage(s, s);
      cp_async_commit();
    }
    for (int kt = 0; kt < KTOT; ++kt) {
      cp_async_wait<ST - 2>();
      __syncthreads();
      const int nk = kt + ST - 1;
      if (nk < KTOT) load_stage(nk % ST, nk);
      cp_async_commit();
      const double2 *as = As + (kt % ST) * A_STAGE;
      const double2 *bs = Bs + (kt % ST) * B_STAGE;
#pragma unroll
      for (int kq = 0; kq < BK / 4; ++kq) {
        double ar[4], ai[4], an[4], br[4], bi[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const double2 a = as[(wm * 32 + i * 8 + (lane >> 2)) * APITCH + kq * 4 + (lane & 3)];
          ar[i] = a.x; ai[i] = a.y; an[i] = dneg(a.y);
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const double2 b = bs[(kq * 4 + (lane & 3)) * BPITCH + wn * 32 + j * 8 + (lane >> 2)];
          br[j] = b.x; bi[j] = b.y;
        }
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            dmma(cr[i][j][0], cr[i][j][1], ar[i], br[j]);
            dmma(ci[i][j][0], ci[i][j][1], ar[i], bi[j]);
            dmma(cr[i][j][0], cr[i][j][1], an[i], bi[j]);
            dmma(ci[i][j][0], ci[i][j][1], ai[i], br[j]);
          }
      }
    }
    cp_async_wait<0>();
    __syncthreads();  // the smem ring is reused by the next tile

    double2 *Cbase = d.C + t * d.sCt + mo * d.sCmo + no * d.sCno;
    const long long sCmi = d.sCmi, sCni = d.sCni;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int m = m0 + wm * 32 + i * 8 + (lane >> 2);
      if (m >= Mi) continue;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int n = n0 + wn * 32 + j * 8 + (lane & 3) * 2;
        double2 *cp = Cbase + (long long)m * sCmi + (long long)n * sCni;
        if (n < Ni) cp[0] = make_double2(cr[i][j][0], ci[i][j][0]);
        if (n + 1 < Ni) cp[sCni] = make_double2(cr[i][j][1], ci[i][j][1]);
      }
    }
  }
}

// ---------------------------------------------------------------- small-tile GEMM (v6)
//
// Latency hidden by warp parallelism instead of ILP: the configuration cuBLAS picks for
// ZGEMM on this part (ncu of cuBLAS: cutlass_80_tensorop_z884gemm_32x32_16x4, 128 threads,
// 92 registers, 3 CTAs/SM → DMMA pipe 99.5% active; profiles/ncu_cublas_r01.txt).  CTA tile
// TBM×TBN complex, 4 warps of (TBM/2)×(TBN/2), BK 16, TST-stage cp.async ring, one tile
// per CTA (many resident CTAs per SM overlap each other's prologue/epilogue).
template <int TBM, int TBN, int TST>
struct SmallCfg {
  static constexpr int BKs = 16;
  static constexpr int AP = BKs + 4;   // [m][k] rows: 320 B ≡ 64 (mod 128)
  static constexpr int BP = TBN + 2;   // [k][n] rows: (TBN+2)·16 B; TBN = 32 → 544 ≡ 32 (mod 128)
  static constexpr int AE = TBM * AP, BE = BKs * BP;
  static constexpr int SMEM = TST * (AE + BE) * 16;
  static constexpr int MI = TBM / 2 / 8, NJ = TBN / 2 / 8;  // 8x8 blocks per warp
};

template <int TBM, int TBN, int TST>
__device__ __forceinline__ void zgemm_small_body(const GemmDesc *__restrict__ descs, int n_desc, long long total) {
  using Cfg = SmallCfg<TBM, TBN, TST>;
  constexpr int BKs = Cfg::BKs, AP = Cfg::AP, BP = Cfg::BP, MI = Cfg::MI, NJ = Cfg::NJ;
  extern __shared__ __align__(128) double2 smem[];
  double2 *As = smem;
  double2 *Bs = smem + TST * Cfg::AE;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int wm = warp >> 1, wn = warp & 1;
  const long long tile = blockIdx.x;
  if (tile >= total) return;
  int lo = 0, hi = n_desc - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (descs[mid].tile_begin <= tile) lo = mid; else hi = mid - 1;
  }
  const GemmDesc &d = descs[lo];
  long long lt = tile - d.tile_begin;
  const int tilesN = d.tilesN, tilesM = d.tilesM;
  const int tn = (int)(lt % tilesN); lt /= tilesN;
  const int tm = (int)(lt % tilesM); lt /= tilesM;
  const int no = (int)(lt % d.No); lt /= d.No;
  const int mo = (int)(lt % d.Mo);
  const long long t = lt / d.Mo;
  const int m0 = tm * TBM, n0 = tn * TBN;
  const int Mi = d.Mi, Ni = d.Ni, Ki = d.Ki;
  const int sAmi = (int)d.sAmi, sAki = (int)d.sAki, sBki = (int)d.sBki, sBni = (int)d.sBni;
  const double2 *Ab = d.A + t * d.sAt + mo * d.sAmo + (long long)m0 * sAmi;
  const double2 *Bb = d.B + t * d.sBt + no * d.sBno + (long long)n0 * sBni;
  const bool akf = sAki == 1, bnf = sBni == 1;
  const int KT = (Ki + BKs - 1) / BKs, KTOT = d.Ko * KT;
  constexpr int AL = TBM * BKs / 128, BL = TBN * BKs / 128;  // copies per thread per stage

  auto load = [&](int slot, int kt) {
    const int ko = kt / KT;
    const int kb = (kt - ko * KT) * BKs;
    const double2 *Ak = Ab + ko * d.sAko + (long long)kb * sAki;
    const double2 *Bk = Bb + ko * d.sBko + (long long)kb * sBki;
    double2 *as = As + slot * Cfg::AE;
    double2 *bs = Bs + slot * Cfg::BE;
#pragma unroll
    for (int j = 0; j < AL; ++j) {
      const int e = tid + 128 * j;
      int m, k;
      if (akf) { k = e & (BKs - 1); m = e / BKs; } else { m = e % TBM; k = e / TBM; }
      const bool v = (m0 + m < Mi) && (kb + k < Ki);
      cp_async16(as + m * AP + k, v ? Ak + m * sAmi + k * sAki : d.A, v);
    }
#pragma unroll
    for (int j = 0; j < BL; ++j) {
      const int e = tid + 128 * j;
      int n, k;
      if (bnf) { n = e % TBN; k = e / TBN; } else { k = e & (BKs - 1); n = e / BKs; }
      const bool v = (n0 + n < Ni) && (kb + k < Ki);
      cp_async16(bs + k * BP + n, v ? Bk + k * sBki + n * sBni : d.B, v);
    }
  };

  double cr[MI][NJ][2], ci[MI][NJ][2];
#pragma unroll
  for (int i = 0; i < MI; ++i)
#pragma unroll
    for (int j = 0; j < NJ; ++j) { cr[i][j][0] = cr[i][j][1] = ci[i][j][0] = ci[i][j][1] = 0.0; }
#pragma unroll
  for (int s = 0; s < TST - 1; ++s) {
    if (s < KTOT) load(s, s);
    cp_async_commit();
  }
  for (int kt = 0; kt < KTOT; ++kt) {
    cp_async_wait<TST - 2>();
    __syncthreads();
    const int nk = kt + TST - 1;
    if (nk < KTOT) load(nk % TST, nk);
    cp_async_commit();
    const double2 *as = As + (kt % TST) * Cfg::AE;
    const double2 *bs = Bs + (kt % TST) * Cfg::BE;
#pragma unroll
    for (int kq = 0; kq < BKs / 4; ++kq) {
      double ar[MI], ai[MI], br[NJ], bi[NJ];
#pragma unroll
      for (int i = 0; i < MI; ++i) {
        const double2 a = as[(wm * MI * 8 + i * 8 + (lane >> 2)) * AP + kq * 4 + (lane & 3)];
        ar[i] = a.x; ai[i] = a.y;
      }
#pragma unroll
      for (int j = 0; j < NJ; ++j) {
        const double2 b = bs[(kq * 4 + (lane & 3)) * BP + wn * NJ * 8 + j * 8 + (lane >> 2)];
        br[j] = b.x; bi[j] = b.y;
      }
#pragma unroll
      for (int i = 0; i < MI; ++i)
#pragma unroll
        for (int j = 0; j < NJ; ++j) {
          dmma(cr[i][j][0], cr[i][j][1], ar[i], br[j]);
          dmma(ci[i][j][0], ci[i][j][1], ar[i], bi[j]);
        }
#pragma unroll
      for (int i = 0; i < MI; ++i)
#pragma unroll
        for (int j = 0; j < NJ; ++j) {
          dmma(cr[i][j][0], cr[i][j][1], dneg(ai[i]), bi[j]);
          dmma(ci[i][j][0], ci[i][j][1], ai[i], br[j]);
        }
    }
  }
  cp_async_wait<0>();
  double2 *C = d.C + t * d.sCt + mo * d.sCmo + no * d.sCno;
  const long long sCmi = d.sCmi, sCni = d.sCni;
#pragma unroll
  for (int i = 0; i < MI; ++i) {
    const int m = m0 + wm * MI * 8 + i * 8 + (lane >> 2);
    if (m >= Mi) continue;
#pragma unroll
    for (int j = 0; j < NJ; ++j) {
      const int n = n0 + wn * NJ * 8 + j * 8 + (lane & 3) * 2;
      double2 *cp = C + (long long)m * sCmi + (long long)n * sCni;
      if (n < Ni) cp[0] = make_double2(cr[i][j][0], ci[i][j][0]);
      if (n + 1 < Ni) cp[sCni] = make_double2(cr[i][j][1], ci[i][j][1]);
    }
  }
}

// ---------------------------------------------------------------- persistent GEMM (v2, 3M)
//
// The production GEMM.  Persistent CTAs (2 per SM) take every G-th tile and run one
// continuous cp.async pipeline (BK = 16, 3 stages) over their whole (tile, k-step) sequence;
// the next stage's copies are issued in NPART pieces inside the DMMA stream of the stage being
// computed so they occupy the DMMA pacing slots; the task descriptor advances linearly.
// Optional fused final dot (GemmDesc::D) in the epilogue.
//
// Complex product, two schemes (template M3):
//   4M (default before round-1 end): Cr += Ar·Br + (−Ai)·Bi, Ci += Ar·Bi + Ai·Br  — 4 DMMAs
//   3M (Gauss): K1 += (Ar+Ai)·Br, K2 += Ar·(Bi−Br), K3 += Ai·(Br+Bi);
//               Cr = K1 − K3, Ci = K1 + K2                                       — 3 DMMAs
// The 3M scheme does 25% fewer DMMAs for the same algorithmic work (8 real flops per complex
// MAC are still what the roofline counts); its rounding differs from the 4M one but stays far
// inside the 1e-10 parity bound, and exact-integer inputs stay bit-exact (every partial sum
// is an integer below 2^53; SURVEY.md §8(c) "Bit-exact GPU parity").
constexpr int BK2 = 16, ST2 = 3;
constexpr int APITCH2 = BK2 + 4;  // [m][k] rows: 320 B ≡ 64 (mod 128): A fragment loads conflict-free

template <int TBM, int TBN>
struct PCfg {
  static constexpr int BP = TBN + 2;  // [k][n] rows: (TBN+2)·16 B ≡ 32 (mod 128) for TBN ∈ {32, 64}
  static constexpr int AE = TBM * APITCH2, BE = BK2 * BP;
  static constexpr int SMEM = ST2 * (AE + BE) * 16;
};
constexpr int GEMM2_SMEM = PCfg<64, 64>::SMEM;

template <int LPTA, int LPTB>
struct LoadCur {
  const double2 *A, *B;  // tile bases (t, mo/no, m0/n0 applied)
  long long sAko, sBko;
  int sAki, sBki;
  int Ki, KT, KTOT;
  int offA[LPTA], offB[LPTB];
  unsigned vA, vB;       // m-valid / n-valid bit per element
  bool akf, bnf;
};

struct StoreCur {
  double2 *C;
  int sCmi, sCni, Mi, Ni, m0, n0, KTOT;
  const double2 *D;  // fused final dot: the partner tile base (nullptr = plain GEMM)
  long long pidx;    // first partial-sum slot of this tile
};

template <int NTH, int TBM, int TBN, int LPTA, int LPTB>
__device__ __forceinline__ void decode_tile(const GemmDesc *__restrict__ descs, int n_desc, int &task,
                                            long long tile, int tid, LoadCur<LPTA, LPTB> *L, StoreCur *S) {
  while (task + 1 < n_desc && descs[task + 1].tile_begin <= tile) ++task;
  const GemmDesc &d = descs[task];
  long long lt = tile - d.tile_begin;
  const int tilesN = d.tilesN, tilesM = d.tilesM, No = d.No, Mo = d.Mo;
  const int tn = (int)(lt % tilesN); lt /= tilesN;
  const int tm = (int)(lt % tilesM); lt /= tilesM;
  const int no = (int)(lt % No); lt /= No;
  const int mo = (int)(lt % Mo);
  const long long t = lt / Mo;
  const int m0 = tm * TBM, n0 = tn * TBN;
  const int KT = (d.Ki + BK2 - 1) / BK2;
  if (L) {
    const int sAmi = (int)d.sAmi, sAki = (int)d.sAki, sBki = (int)d.sBki, sBni = (int)d.sBni;
    L->A = d.A + t * d.sAt + mo * d.sAmo + (long long)m0 * sAmi;
    L->B = d.B + t * d.sBt + no * d.sBno + (long long)n0 * sBni;
    L->sAko = d.sAko; L->sBko = d.sBko; L->sAki = sAki; L->sBki = sBki;
    L->Ki = d.Ki; L->KT = KT; L->KTOT = d.Ko * KT;
    L->akf = (sAki == 1);
    L->bnf = (sBni == 1);
    const int Mi = d.Mi, Ni = d.Ni;
    L->vA = 0; L->vB = 0;
#pragma unroll
    for (int j = 0; j < LPTA; ++j) {
      const int e = tid + j * NTH;
      int m, k;
      if (L->akf) { k = e & (BK2 - 1); m = e / BK2; } else { m = e % TBM; k = e / TBM; }
      L->offA[j] = m * sAmi + k * sAki;
      if (m0 + m < Mi) L->vA |= 1u << j;
    }
#pragma unroll
    for (int j = 0; j < LPTB; ++j) {
      const int e = tid + j * NTH;
      int n, kb;
      if (L->bnf) { n = e % TBN; kb = e / TBN; } else { kb = e & (BK2 - 1); n = e / BK2; }
      L->offB[j] = kb * sBki + n * sBni;
      if (n0 + n < Ni) L->vB |= 1u << j;
    }
  }
  if (S) {
    S->C = d.C + t * d.sCt + mo * d.sCmo + no * d.sCno;
    S->sCmi = (int)d.sCmi; S->sCni = (int)d.sCni;
    S->Mi = d.Mi; S->Ni = d.Ni; S->m0 = m0; S->n0 = n0;
    S->KTOT = d.Ko * KT;
    S->D = d.D ? d.D + t * d.sDt + mo * d.sDmo + no * d.sDno : nullptr;
    S->pidx = (tile - d.tile_begin) * (NTH / 32);
  }
}

// NWM × NWN warps with WTM × WTN complex warp tiles; CTA tile (NWM·WTM) × (NWN·WTN).
template <int NWM, int NWN, int WTM, int WTN, bool M3>
__device__ __forceinline__ void zgemm_persistent_body(const GemmDesc *__restrict__ descs, int n_desc,
                                                      long long total) {
  constexpr int NTH = NWM * NWN * 32;
  constexpr int TBM = NWM * WTM, TBN = NWN * WTN;
  constexpr int LPTA = (TBM * BK2) / NTH, LPTB = (TBN * BK2) / NTH;
  constexpr int MI = WTM / 8, NJ = WTN / 8;  // 8x8 blocks per warp
  constexpr int NACC = M3 ? 3 : 2;
  using Cfg = PCfg<TBM, TBN>;
  constexpr int BP = Cfg::BP;
  extern __shared__ __align__(128) double2 smem[];
  double2 *As = smem;
  double2 *Bs = smem + ST2 * Cfg::AE;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int wm = warp / NWN, wn = warp % NWN;

  // CTA c takes tiles c, c + G, c + 2G, ...: the CTAs running at any moment work on
  // neighbouring tiles (the same slices), so each A/B block is fetched from DRAM once and
  // served to the other CTAs from L2 (contiguous per-CTA ranges doubled the DRAM reads)
  const long long G = gridDim.x, t_begin = blockIdx.x;
  if (t_begin >= total) return;

  int task_l = 0, task_c = 0;
  {  // first task by binary search, then linear advance
    int lo = 0, hi = n_desc - 1;
    while (lo < hi) {
      int mid = (lo + hi + 1) >> 1;
      if (descs[mid].tile_begin <= t_begin) lo = mid; else hi = mid - 1;
    }
    task_l = task_c = lo;
  }
  LoadCur<LPTA, LPTB> L;
  StoreCur S;
  long long tile_l = t_begin, tile_c = t_begin;
  int kt_l = 0, kt_c = 0;
  decode_tile<NTH, TBM, TBN, LPTA, LPTB>(descs, n_desc, task_l, tile_l, tid, &L, nullptr);
  decode_tile<NTH, TBM, TBN, LPTA, LPTB>(descs, n_desc, task_c, tile_c, tid, (LoadCur<LPTA, LPTB> *)nullptr, &S);
  bool more_l = true;

  // The loads of a stage are issued in NPART pieces interleaved with the DMMA stream of the
  // stage being computed (one piece per k-quad), so the scheduler can slot the cp.async and
  // address arithmetic into the DMMA pacing gaps instead of running a separate load phase.
  constexpr int NPART = BK2 / 4;
  static_assert(LPTA % NPART == 0 && LPTB % NPART == 0, "load split");
  const double2 *ldA = nullptr, *ldB = nullptr;
  int ld_kb = 0;
  auto begin_load = [&]() {
    const int ko = kt_l / L.KT;
    ld_kb = (kt_l - ko * L.KT) * BK2;
    ldA = L.A + ko * L.sAko + (long long)ld_kb * L.sAki;
    ldB = L.B + ko * L.sBko + (long long)ld_kb * L.sBki;
  };
  auto issue_part = [&](int slot, int part) {
    double2 *as = As + slot * Cfg::AE;
    double2 *bs = Bs + slot * Cfg::BE;
#pragma unroll
    for (int jj = 0; jj < LPTA / NPART; ++jj) {
      const int j = part * (LPTA / NPART) + jj;
      const int e = tid + j * NTH;
      int m, k;
      if (L.akf) { k = e & (BK2 - 1); m = e / BK2; } else { m = e % TBM; k = e / TBM; }
      const bool v = ((L.vA >> j) & 1u) && (ld_kb + k < L.Ki);
      cp_async16(as + m * APITCH2 + k, v ? ldA + L.offA[j] : L.A, v);
    }
#pragma unroll
    for (int jj = 0; jj < LPTB / NPART; ++jj) {
      const int j = part * (LPTB / NPART) + jj;
      const int e = tid + j * NTH;
      int n, k;
      if (L.bnf) { n = e % TBN; k = e / TBN; } else { k = e & (BK2 - 1); n = e / BK2; }
      const bool v = ((L.vB >> j) & 1u) && (ld_kb + k < L.Ki);
      cp_async16(bs + k * BP + n, v ? ldB + L.offB[j] : L.B, v);
    }
  };
  auto advance_load = [&]() {  // next k-step, possibly in the next tile
    if (++kt_l == L.KTOT) {
      kt_l = 0;
      if ((tile_l += G) < total) decode_tile<NTH, TBM, TBN, LPTA, LPTB>(descs, n_desc, task_l, tile_l, tid, &L, nullptr);
      else more_l = false;
    }
  };
  auto issue_load = [&](int slot) {
    begin_load();
#pragma unroll
    for (int p = 0; p < NPART; ++p) issue_part(slot, p);
    advance_load();
  };

  double acc[MI][NJ][NACC][2];
#pragma unroll
  for (int i = 0; i < MI; ++i)
#pragma unroll
    for (int j = 0; j < NJ; ++j)
#pragma unroll
      for (int q = 0; q < NACC; ++q) acc[i][j][q][0] = acc[i][j][q][1] = 0.0;

#pragma unroll
  for (int s = 0; s < ST2 - 1; ++s) {
    if (more_l) issue_load(s);
    cp_async_commit();
  }
  int slot_c = 0, slot_l = ST2 - 1;
  for (;;) {
    cp_async_wait<ST2 - 2>();
    __syncthreads();
    const bool ld = more_l;
    if (ld) begin_load();
    const double2 *as = As + slot_c * Cfg::AE;
    const double2 *bs = Bs + slot_c * Cfg::BE;
    // Fragments are double-buffered inside the stage: the LDS (and, for 3M, the operand
    // sums on the FP64 pipe) of k-quad q+1 are issued before the DMMAs of q, so neither
    // the shared-memory latency nor a DADD waiting behind DMMAs sits in front of them.
    constexpr int FA = M3 ? 3 : 2, FB = M3 ? 3 : 2;
    double fa[2][MI][FA], fb[2][NJ][FB];
    auto load_frag = [&](int buf, int kq) {
#pragma unroll
      for (int i = 0; i < MI; ++i) {
        const double2 a = as[(wm * WTM + i * 8 + (lane >> 2)) * APITCH2 + kq * 4 + (lane & 3)];
        fa[buf][i][0] = a.x;
        fa[buf][i][1] = a.y;
        if constexpr (M3) fa[buf][i][2] = a.x + a.y;  // Ar + Ai
      }
#pragma unroll
      for (int j = 0; j < NJ; ++j) {
        const double2 b = bs[(kq * 4 + (lane & 3)) * BP + wn * WTN + j * 8 + (lane >> 2)];
        fb[buf][j][0] = b.x;
        fb[buf][j][1] = b.y;
        if constexpr (M3) {
          fb[buf][j][1] = b.y - b.x;  // Bi − Br
          fb[buf][j][2] = b.x + b.y;  // Br + Bi
        }
      }
    };
    // (4M keeps a single buffer: its 128 accumulator registers leave no room for a second)
    if constexpr (M3) load_frag(0, 0);
#pragma unroll
    for (int kq = 0; kq < BK2 / 4; ++kq) {
      if (ld) issue_part(slot_l, kq);
      const int cur = M3 ? (kq & 1) : 0;
      if constexpr (M3) {
        if (kq + 1 < BK2 / 4) load_frag(cur ^ 1, kq + 1);
      } else {
        load_frag(0, kq);
      }
      if constexpr (M3) {
#pragma unroll
        for (int i = 0; i < MI; ++i)
#pragma unroll
          for (int j = 0; j < NJ; ++j) {
            dmma(acc[i][j][0][0], acc[i][j][0][1], fa[cur][i][2], fb[cur][j][0]);  // (Ar+Ai)·Br
            dmma(acc[i][j][1][0], acc[i][j][1][1], fa[cur][i][0], fb[cur][j][1]);  // Ar·(Bi−Br)
            dmma(acc[i][j][2][0], acc[i][j][2][1], fa[cur][i][1], fb[cur][j][2]);  // Ai·(Br+Bi)
          }
      } else {
#pragma unroll
        for (int i = 0; i < MI; ++i)
#pragma unroll
          for (int j = 0; j < NJ; ++j) {
            dmma(acc[i][j][0][0], acc[i][j][0][1], fa[cur][i][0], fb[cur][j][0]);
            dmma(acc[i][j][1][0], acc[i][j][1][1], fa[cur][i][0], fb[cur][j][1]);
          }
#pragma unroll
        for (int i = 0; i < MI; ++i)
#pragma unroll
          for (int j = 0; j < NJ; ++j) {
            dmma(acc[i][j][0][0], acc[i][j][0][1], dneg(fa[cur][i][1]), fb[cur][j][1]);
            dmma(acc[i][j][1][0], acc[i][j][1][1], fa[cur][i][1], fb[cur][j][0]);
          }
      }
    }
    if (ld) advance_load();
    cp_async_commit();
    slot_l = (slot_l + 1 == ST2) ? 0 : slot_l + 1;
    slot_c = (slot_c + 1 == ST2) ? 0 : slot_c + 1;
    if (S.D && kt_c + 2 == S.KTOT) {
      // fused dot: pull this tile's partner block into L2 one k-step before the epilogue
      const GemmDesc &dd = descs[task_c];
      const bool mrow = dd.sDni == 1;  // contiguous runs along n (else along m, sDmi == 1)
      const int rows = mrow ? min(TBM, S.Mi - S.m0) : min(TBN, S.Ni - S.n0);
      const int segs = (mrow ? TBN : TBM) / 8;
      for (int q = tid; q < rows * segs; q += NTH) {
        const int r = q / segs, seg = (q % segs) * 8;
        const double2 *pp = mrow ? S.D + (long long)(S.m0 + r) * dd.sDmi + S.n0 + seg
                                 : S.D + (long long)(S.n0 + r) * dd.sDni + S.m0 + seg;
        asm volatile("prefetch.global.L2 [%0];\n" ::"l"(pp));
      }
    }
    if (++kt_c == S.KTOT) {  // tile done: write back (next tile's loads already in flight)
      // the complex value of accumulator block (i, j), half h
      auto cval = [&](int i, int j, int h, double &re, double &im) {
        if constexpr (M3) {
          re = acc[i][j][0][h] - acc[i][j][2][h];
          im = acc[i][j][0][h] + acc[i][j][1][h];
        } else {
          re = acc[i][j][0][h];
          im = acc[i][j][1][h];
        }
      };
      if (S.D) {
        // fused final contraction: this warp's partial Σ C·D (no C written)
        const GemmDesc &dd = descs[task_c];
        const long long sDmi = dd.sDmi, sDni = dd.sDni;
        double pr = 0.0, pim = 0.0;
#pragma unroll
        for (int i = 0; i < MI; ++i) {
          const int m = S.m0 + wm * WTM + i * 8 + (lane >> 2);
          double2 y[NJ][2];
#pragma unroll
          for (int j = 0; j < NJ; ++j)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              const int n = S.n0 + wn * WTN + j * 8 + (lane & 3) * 2 + h;
              y[j][h] = (m < S.Mi && n < S.Ni) ? S.D[(long long)m * sDmi + (long long)n * sDni] : make_double2(0.0, 0.0);
            }
#pragma unroll
          for (int j = 0; j < NJ; ++j)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              double re, im;
              cval(i, j, h, re, im);
              pr += re * y[j][h].x - im * y[j][h].y;
              pim += re * y[j][h].y + im * y[j][h].x;
            }
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) {
          pr += __shfl_xor_sync(0xffffffffu, pr, off);
          pim += __shfl_xor_sync(0xffffffffu, pim, off);
        }
        if (lane == 0) dd.part[S.pidx + warp] = make_double2(pr, pim);
      } else {
#pragma unroll
        for (int i = 0; i < MI; ++i) {
          const int m = S.m0 + wm * WTM + i * 8 + (lane >> 2);
#pragma unroll
          for (int j = 0; j < NJ; ++j) {
            const int n = S.n0 + wn * WTN + j * 8 + (lane & 3) * 2;
            if (m < S.Mi) {
              double re, im;
              double2 *cp = S.C + (long long)m * S.sCmi + (long long)n * S.sCni;
              cval(i, j, 0, re, im);
              if (n < S.Ni) cp[0] = make_double2(re, im);
              cval(i, j, 1, re, im);
              if (n + 1 < S.Ni) cp[S.sCni] = make_double2(re, im);
            }
          }
        }
      }
#pragma unroll
      for (int i = 0; i < MI; ++i)
#pragma unroll
        for (int j = 0; j < NJ; ++j)
#pragma unroll
          for (int q = 0; q < NACC; ++q) acc[i][j][q][0] = acc[i][j][q][1] = 0.0;
      kt_c = 0;
      if ((tile_c += G) >= total) break;
      decode_tile<NTH, TBM, TBN, LPTA, LPTB>(descs, n_desc, task_c, tile_c, tid, (LoadCur<LPTA, LPTB> *)nullptr, &S);
    }
  }
  cp_async_wait<0>();
}

// ---------------------------------------------------------------- warp-specialized GEMM (v3)
//
// Producer/consumer split so the DMMA warps execute nothing but shared-memory fragment loads
// and DMMAs (the v1/v2 captures show long-scoreboard stalls from the cp.async address math
// and register reuse inside the DMMA warps):
//  * warp 4 (producer) streams tile rows with 1-D bulk async copies
//    (cp.async.bulk ... mbarrier::complete_tx, SASS UBLKCP) into padded shared-memory rows,
//    zero-filling ragged rows/tails itself, and signals a "full" mbarrier per stage;
//  * warps 0-3 (consumers) wait on "full", run the 32×32-complex DMMA warp tiles, release
//    the stage on an "empty" mbarrier, and write C from registers at the end of each tile;
//  * persistent CTAs over contiguous tile ranges; the pipeline runs across tile boundaries.
// The smem orientation follows the global one (A [m][k] or [k][m], B [k][n] or [n][k]) so
// every bulk copy is a contiguous run; the fragment loads are specialised per orientation
// (all four are bank-conflict free with the pitches below).  Operands with no unit-stride
// inner index use zgemm_dmma_kernel.

constexpr int NCW = 4;                    // consumer warps
constexpr int NPW = 4;                    // producer warps (outstanding cp.async spread over 128 lanes)
constexpr int NT3 = (NCW + NPW) * 32;
constexpr int PITCH_MK = BK2 + 4;         // [m][k] / [n][k]: 320 B rows
constexpr int PITCH_KM = BM + 2;          // [k][m] / [k][n]: 1056 B rows

template <bool A_MK, bool B_KN>
struct V3Cfg {
  static constexpr int A_ELEMS = A_MK ? BM * PITCH_MK : BK2 * PITCH_KM;
  static constexpr int B_ELEMS = B_KN ? BK2 * PITCH_KM : BN * PITCH_MK;
  static constexpr int STAGE = A_ELEMS + B_ELEMS;
  static constexpr int ST = (220 * 1024) / (STAGE * 16) > 6 ? 6 : (220 * 1024) / (STAGE * 16);
  static constexpr int SMEM = ST * STAGE * 16 + 2 * ST * 8;
};

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  uint32_t done;
  do {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(bar), "r"(parity)
        : "memory");
  } while (!done);
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("{\n .reg .b64 st;\n mbarrier.arrive.shared::cta.b64 st, [%0];\n}\n" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("{\n .reg .b64 st;\n mbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n}\n" ::"r"(bar),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(bar)
               : "memory");
}

struct V3Tile {  // what both roles need about one tile
  const GemmDesc *d;
  long long t;
  int mo, no, m0, n0, KT, KTOT;
};

__device__ __forceinline__ void v3_decode(const GemmDesc *__restrict__ descs, int n_desc, int &task, long long tile,
                                          V3Tile &T) {
  while (task + 1 < n_desc && descs[task + 1].tile_begin <= tile) ++task;
  const GemmDesc *d = descs + task;
  long long lt = tile - d->tile_begin;
  const int tilesN = d->tilesN, tilesM = d->tilesM, No = d->No, Mo = d->Mo;
  const int tn = (int)(lt % tilesN); lt /= tilesN;
  const int tm = (int)(lt % tilesM); lt /= tilesM;
  T.no = (int)(lt % No); lt /= No;
  T.mo = (int)(lt % Mo);
  T.t = lt / Mo;
  T.m0 = tm * BM;
  T.n0 = tn * BN;
  T.d = d;
  T.KT = (d->Ki + BK2 - 1) / BK2;
  T.KTOT = d->Ko * T.KT;
}

template <bool A_MK, bool B_KN>
__device__ __forceinline__ void zgemm_dmma_ws_body(const GemmDesc *__restrict__ descs, int n_desc, long long total) {
  using Cfg = V3Cfg<A_MK, B_KN>;
  constexpr int ST3 = Cfg::ST;
  extern __shared__ __align__(128) double2 smem[];
  uint64_t *bars = reinterpret_cast<uint64_t *>(smem + ST3 * Cfg::STAGE);  // full[ST3], empty[ST3]
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;

  const long long per = total / gridDim.x, rem = total % gridDim.x;
  const long long t_begin = blockIdx.x * per + min((long long)blockIdx.x, rem);
  const long long t_end = t_begin + per + ((long long)blockIdx.x < rem ? 1 : 0);
  if (t_begin >= t_end) return;
  int task = 0;
  {
    int lo = 0, hi = n_desc - 1;
    while (lo < hi) {
      int mid = (lo + hi + 1) >> 1;
      if (descs[mid].tile_begin <= t_begin) lo = mid; else hi = mid - 1;
    }
    task = lo;
  }
  if (tid == 0) {
    for (int s = 0; s < ST3; ++s) {
      mbar_init(smem_u32(&bars[s]), 32 * NPW);
      mbar_init(smem_u32(&bars[ST3 + s]), NCW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();

  if (warp < NPW) {
    // ------------------------------------------------------------ producer warps
    // Warp 0 on purpose: the SMSP arbiter favours the highest warp id, so the DMMA warp that
    // shares this SMSP (warp 4) wins every issue slot it can use and the producer fills the
    // cycles between its DMMAs (with the producer as warp 4 the CTA ran at the pace of the
    // starved consumer: 65% DMMA-pipe activity, profiles/ncu_gemm_r01_v4.json).
    // Per-thread 16-byte cp.async (LDGSTS) along the unit-stride index of each operand (the
    // bulk-copy variant serialised one UBLKCP per row through the uniform datapath and could
    // not keep up), zero-fill by src-size 0 for ragged rows/tails, and completion signalled
    // to the stage's "full" mbarrier by cp.async.mbarrier.arrive.noinc from every lane.
    int step = 0;
    for (long long tile = t_begin; tile < t_end; ++tile) {
      V3Tile T;
      v3_decode(descs, n_desc, task, tile, T);
      const GemmDesc &d = *T.d;
      const int Ki = d.Ki;
      const long long sAmi = d.sAmi, sAki = d.sAki, sBki = d.sBki, sBni = d.sBni;
      const double2 *Ab = d.A + T.t * d.sAt + T.mo * d.sAmo + (long long)T.m0 * sAmi;
      const double2 *Bb = d.B + T.t * d.sBt + T.no * d.sBno + (long long)T.n0 * sBni;
      const int mv = min(BM, d.Mi - T.m0), nv = min(BN, d.Ni - T.n0);  // valid rows / cols
      for (int kt = 0; kt < T.KTOT; ++kt, ++step) {
        const int slot = step % ST3;
        const uint32_t full = smem_u32(&bars[slot]), empty = smem_u32(&bars[ST3 + slot]);
        mbar_wait(empty, ((step / ST3) & 1) ^ 1);
        const int ko = kt / T.KT;
        const int kb = (kt - ko * T.KT) * BK2;
        const int kv = min(BK2, Ki - kb);  // valid k in this step
        const double2 *Ak = Ab + ko * d.sAko + (long long)kb * sAki;
        const double2 *Bk = Bb + ko * d.sBko + (long long)kb * sBki;
        double2 *as = smem + slot * Cfg::STAGE;
        double2 *bs = as + Cfg::A_ELEMS;
#pragma unroll 4
        for (int j = 0; j < (BM * BK2) / (32 * NPW); ++j) {
          const int e = tid + 32 * NPW * j;
          int m, k;
          if (A_MK) { k = e & (BK2 - 1); m = e / BK2; } else { m = e & (BM - 1); k = e / BM; }
          const bool v = m < mv && k < kv;
          const double2 *src = v ? Ak + m * sAmi + k * sAki : d.A;
          cp_async16(A_MK ? as + m * PITCH_MK + k : as + k * PITCH_KM + m, src, v);
        }
#pragma unroll 4
        for (int j = 0; j < (BN * BK2) / (32 * NPW); ++j) {
          const int e = tid + 32 * NPW * j;
          int n, k;
          if (B_KN) { n = e & (BN - 1); k = e / BN; } else { k = e & (BK2 - 1); n = e / BK2; }
          const bool v = n < nv && k < kv;
          const double2 *src = v ? Bk + k * sBki + n * sBni : d.B;
          cp_async16(B_KN ? bs + k * PITCH_KM + n : bs + n * PITCH_MK + k, src, v);
        }
        asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];\n" ::"r"(full) : "memory");
      }
    }
    asm volatile("cp.async.wait_all;\n" ::: "memory");
    return;
  }

  // -------------------------------------------------------------- consumer warps
  // One consumer warp per SMSP: it must issue a DMMA every 16 cycles, so its shared-memory
  // fragment loads for k-quad q+1 are issued before the DMMAs of q (double-buffered
  // fragments), and the next stage is awaited one k-quad early.
  const int cw = warp - NPW;  // consumer index 0..3
  const int wm = cw >> 1, wn = cw & 1;
  double cr[4][4][2], ci[4][4][2];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) { cr[i][j][0] = cr[i][j][1] = ci[i][j][0] = ci[i][j][1] = 0.0; }
  double fa[2][4][2], fb[2][4][2];  // [buffer][i or j][re, im]
  auto load_frags = [&](int buf, const double2 *as, const double2 *bs, int kq) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int m = wm * 32 + i * 8 + (lane >> 2), k = kq * 4 + (lane & 3);
      const double2 a = A_MK ? as[m * PITCH_MK + k] : as[k * PITCH_KM + m];
      fa[buf][i][0] = a.x; fa[buf][i][1] = a.y;
    }
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int n = wn * 32 + j * 8 + (lane >> 2), k = kq * 4 + (lane & 3);
      const double2 b = B_KN ? bs[k * PITCH_KM + n] : bs[n * PITCH_MK + k];
      fb[buf][j][0] = b.x; fb[buf][j][1] = b.y;
    }
  };
  auto mma_quad = [&](int buf) {
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        dmma(cr[i][j][0], cr[i][j][1], fa[buf][i][0], fb[buf][j][0]);
        dmma(ci[i][j][0], ci[i][j][1], fa[buf][i][0], fb[buf][j][1]);
      }
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        dmma(cr[i][j][0], cr[i][j][1], dneg(fa[buf][i][1]), fb[buf][j][1]);
        dmma(ci[i][j][0], ci[i][j][1], fa[buf][i][1], fb[buf][j][0]);
      }
  };
  // the whole CTA range is one sequence of k-steps; count them
  int step = 0;
  V3Tile T;
  long long tile = t_begin;
  v3_decode(descs, n_desc, task, tile, T);
  int kt = 0;
  mbar_wait(smem_u32(&bars[0]), 0);
  load_frags(0, smem, smem + Cfg::A_ELEMS, 0);
  for (;;) {
    const int slot = step % ST3;
    const double2 *as = smem + slot * Cfg::STAGE;
    const double2 *bs = as + Cfg::A_ELEMS;
    // is there a next k-step (this tile or the next)?
    const bool last_k = (kt + 1 == T.KTOT);
    const bool has_next = !last_k || (tile + 1 < t_end);
    const int nslot = (slot + 1 == ST3) ? 0 : slot + 1;
    const double2 *nas = smem + nslot * Cfg::STAGE;
#pragma unroll
    for (int kq = 0; kq < BK2 / 4; ++kq) {
      const int cur = kq & 1;
      if (kq + 1 < BK2 / 4) {
        load_frags(cur ^ 1, as, bs, kq + 1);
      } else if (has_next) {
        mbar_wait(smem_u32(&bars[nslot]), ((step + 1) / ST3) & 1);
        load_frags(cur ^ 1, nas, nas + Cfg::A_ELEMS, 0);
      }
      if (kq + 1 == BK2 / 4) {  // every fragment of this stage is in registers: release it
        __syncwarp();
        if (lane == 0) mbar_arrive(smem_u32(&bars[ST3 + slot]));
      }
      mma_quad(cur);
    }
    ++step;
    if (!last_k) { ++kt; continue; }
    // tile done: epilogue from registers (the producer keeps filling the next stages)
    if (T.d->D) {  // fused final contraction: partial Σ C·D of this warp's 32×32 block
      const GemmDesc &d = *T.d;
      const double2 *Dp = d.D + T.t * d.sDt + T.mo * d.sDmo + T.no * d.sDno;
      const long long sDmi = d.sDmi, sDni = d.sDni;
      const int Mi = d.Mi, Ni = d.Ni;
      double pr = 0.0, pim = 0.0;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int m = T.m0 + wm * 32 + i * 8 + (lane >> 2);
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const int n = T.n0 + wn * 32 + j * 8 + (lane & 3) * 2;
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            if (m < Mi && n + h < Ni) {
              const double2 y = Dp[(long long)m * sDmi + (long long)(n + h) * sDni];
              pr += cr[i][j][h] * y.x - ci[i][j][h] * y.y;
              pim += cr[i][j][h] * y.y + ci[i][j][h] * y.x;
            }
          }
          cr[i][j][0] = cr[i][j][1] = ci[i][j][0] = ci[i][j][1] = 0.0;
        }
      }
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        pr += __shfl_xor_sync(0xffffffffu, pr, off);
        pim += __shfl_xor_sync(0xffffffffu, pim, off);
      }
      if (lane == 0) d.part[(tile - d.tile_begin) * NCW + cw] = make_double2(pr, pim);
    } else {
      const GemmDesc &d = *T.d;
      double2 *C = d.C + T.t * d.sCt + T.mo * d.sCmo + T.no * d.sCno;
      const long long sCmi = d.sCmi, sCni = d.sCni;
      const int Mi = d.Mi, Ni = d.Ni;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int m = T.m0 + wm * 32 + i * 8 + (lane >> 2);
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const int n = T.n0 + wn * 32 + j * 8 + (lane & 3) * 2;
          if (m < Mi) {
            double2 *cp = C + (long long)m * sCmi + (long long)n * sCni;
            if (n < Ni) cp[0] = make_double2(cr[i][j][0], ci[i][j][0]);
            if (n + 1 < Ni) cp[sCni] = make_double2(cr[i][j][1], ci[i][j][1]);
          }
          cr[i][j][0] = cr[i][j][1] = ci[i][j][0] = ci[i][j][1] = 0.0;
        }
      }
    }
    if (++tile >= t_end) break;
    v3_decode(descs, n_desc, task, tile, T);
    kt = 0;
  }
}

// ---------------------------------------------------------------- dot / trace

constexpr int DT = 256;

__device__ __forceinline__ void cmac(double &sr, double &si, double2 a, double2 b) {
  sr += a.x * b.x - a.y * b.y;
  si += a.x * b.y + a.y * b.x;
}

constexpr int DOT_SMEM = 2 * 32 * 33 * 16;  // two 32×33 complex tiles (33.8 KB)

__device__ __forceinline__ void zdot_body(const DotDesc *__restrict__ descs, int n_desc) {
  extern __shared__ __align__(16) double2 dsm[];
  __shared__ double red[2][DT / 32];
  const long long cta = blockIdx.x;
  int lo = 0, hi = n_desc - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (descs[mid].cta_begin <= cta) lo = mid; else hi = mid - 1;
  }
  const DotDesc &d = descs[lo];
  const int t = (int)(cta - d.cta_begin);
  const int tid = threadIdx.x;
  const double2 *A = d.A + t * d.sAt;
  const double2 *B = d.B ? d.B + t * d.sBt : nullptr;
  double sr = 0.0, si = 0.0;
  const long long O0 = d.O[0], O1 = d.O[1], O2 = d.O[2];
  const long long Ototal = O0 * O1 * O2;
  if (d.mode == 3) {
    for (int i = tid; i < d.X; i += DT) {
      const double2 a = A[i];
      sr += a.x;
      si += a.y;
    }
  } else if (d.mode == 2) {
    for (int i = tid; i < d.X; i += DT) {
      const double2 a = A[(long long)i * d.sAx];
      sr += a.x;
      si += a.y;
    }
  } else if (d.mode == 0) {
    const long long X = d.X, total = Ototal * X;
#pragma unroll 4
    for (long long e = tid; e < total; e += DT) {
      const long long o = e / X, x = e - o * X;
      const long long o2 = o % O2, o01 = o / O2, o1 = o01 % O1, o0 = o01 / O1;
      const long long offA = o0 * d.sAo[0] + o1 * d.sAo[1] + o2 * d.sAo[2] + x * d.sAx;
      const long long offB = o0 * d.sBo[0] + o1 * d.sBo[1] + o2 * d.sBo[2] + x * d.sBx;
      cmac(sr, si, A[offA], B[offB]);
    }
  } else {  // transpose tiles: A contiguous along x, B contiguous along y (32×32 smem tiles)
    double2 (*As)[33] = reinterpret_cast<double2 (*)[33]>(dsm);
    double2 (*Bs)[33] = reinterpret_cast<double2 (*)[33]>(dsm + 32 * 33);
    const int ty = tid >> 5, tx = tid & 31;
    for (long long o = 0; o < Ototal; ++o) {
      const long long o2 = o % O2, o01 = o / O2, o1 = o01 % O1, o0 = o01 / O1;
      const double2 *Ao = A + o0 * d.sAo[0] + o1 * d.sAo[1] + o2 * d.sAo[2];
      const double2 *Bo = B + o0 * d.sBo[0] + o1 * d.sBo[1] + o2 * d.sBo[2];
      for (int y0 = 0; y0 < d.Y; y0 += 32)
        for (int x0 = 0; x0 < d.X; x0 += 32) {
          for (int r = ty; r < 32; r += DT / 32) {
            const int y = y0 + r, x = x0 + tx;
            As[r][tx] = (y < d.Y && x < d.X) ? Ao[(long long)y * d.sAy + (long long)x * d.sAx] : make_double2(0, 0);
            const int xb = x0 + r, yb = y0 + tx;
            Bs[r][tx] = (xb < d.X && yb < d.Y) ? Bo[(long long)xb * d.sBx + (long long)yb * d.sBy] : make_double2(0, 0);
          }
          __syncthreads();
          for (int r = ty; r < 32; r += DT / 32) cmac(sr, si, As[r][tx], Bs[tx][r]);
          __syncthreads();
        }
    }
  }
  // deterministic block reduction: xor butterfly, then warps in order
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    sr += __shfl_xor_sync(0xffffffffu, sr, off);
    si += __shfl_xor_sync(0xffffffffu, si, off);
  }
  if ((tid & 31) == 0) { red[0][tid >> 5] = sr; red[1][tid >> 5] = si; }
  __syncthreads();
  if (tid == 0) {
    double ar = 0.0, ai = 0.0;
    for (int w = 0; w < DT / 32; ++w) { ar += red[0][w]; ai += red[1][w]; }
    d.out[t] = make_double2(ar, ai);
  }
}

// ---------------------------------------------------------------- finalize / sum

__global__ void finalize_kernel(int G, int Lt, const int *__restrict__ comp_off,
                                const int *__restrict__ comp_slot, const double2 *__restrict__ S,
                                double2 *__restrict__ vals) {
  const long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  if (i >= (long long)G * Lt) return;
  const int g = (int)(i / Lt), t = (int)(i % Lt);
  double vr = 1.0, vi = 0.0;
  for (int c = comp_off[g]; c < comp_off[g + 1]; ++c) {
    const double2 s = S[(long long)comp_slot[c] * Lt + t];
    const double nr = vr * s.x - vi * s.y, ni = vr * s.y + vi * s.x;
    vr = nr;
    vi = ni;
  }
  vals[i] = make_double2(vr, vi);
}

__global__ void __launch_bounds__(DT) corr_sum_kernel(int G, int Lt, const double2 *__restrict__ coefs,
                                                      const double2 *__restrict__ vals,
                                                      double2 *__restrict__ corr) {
  __shared__ double red[2][DT / 32];
  const int t = blockIdx.x, tid = threadIdx.x;
  double sr = 0.0, si = 0.0;
  for (int g = tid; g < G; g += DT) {
    const double2 c = coefs[g], v = vals[(long long)g * Lt + t];
    sr += c.x * v.x - c.y * v.y;
    si += c.x * v.y + c.y * v.x;
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    sr += __shfl_xor_sync(0xffffffffu, sr, off);
    si += __shfl_xor_sync(0xffffffffu, si, off);
  }
  if ((tid & 31) == 0) { red[0][tid >> 5] = sr; red[1][tid >> 5] = si; }
  __syncthreads();
  if (tid == 0) {
    double ar = 0.0, ai = 0.0;
    for (int w = 0; w < DT / 32; ++w) { ar += red[0][w]; ai += red[1][w]; }
    corr[t] = make_double2(ar, ai);
  }
}

__global__ void accumulate_kernel(double2 *dst, const double2 *src, long long n) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
       i += (long long)gridDim.x * blockDim.x) {
    const double2 a = dst[i], b = src[i];
    dst[i] = make_double2(a.x + b.x, a.y + b.y);
  }
}


// Kernel entry points.  Descriptors travel as __grid_constant__ kernel parameters (up to
// 32 KB per launch on sm_100): no H2D memcpy on the compute stream, which would otherwise
// queue behind the node prefetch copies on the copy engine and serialise compute behind H2D.
__global__ void __launch_bounds__(NT, 2) zgemm_dmma_kernel(const __grid_constant__ GemmBatch b, long long total) {
  zgemm_dmma_kernel_body(b.d, b.n, total);
}
template <int TBM, int TBN, int TST, int MINB>
__global__ void __launch_bounds__(128, MINB) zgemm_small(const __grid_constant__ GemmBatch b, long long total) {
  zgemm_small_body<TBM, TBN, TST>(b.d, b.n, total);
}
template <int NWM, int NWN, int WTM, int WTN, bool M3>
__global__ void __launch_bounds__(NWM * NWN * 32, 2)
    zgemm_persistent(const __grid_constant__ GemmBatch b, long long total) {
  zgemm_persistent_body<NWM, NWN, WTM, WTN, M3>(b.d, b.n, total);
}
template <int NWM, int NWN, int WTM, int WTN, bool M3>
__global__ void __launch_bounds__(NWM * NWN * 32, 1)
    zgemm_persistent1(const __grid_constant__ GemmBatch b, long long total) {
  zgemm_persistent_body<NWM, NWN, WTM, WTN, M3>(b.d, b.n, total);
}
template <bool A_MK, bool B_KN>
__global__ void __launch_bounds__(NT3, 1) zgemm_dmma_ws(const __grid_constant__ GemmBatch b, long long total) {
  zgemm_dmma_ws_body<A_MK, B_KN>(b.d, b.n, total);
}
__global__ void __launch_bounds__(DT) zdot_kernel(const __grid_constant__ DotBatch b) { zdot_body(b.d, b.n); }

template <bool A_MK, bool B_KN>
cudaError_t launch_ws(const GemmBatch *b, long long total, int sms, cudaStream_t st) {
  using Cfg = V3Cfg<A_MK, B_KN>;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(zgemm_dmma_ws<A_MK, B_KN>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         Cfg::SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  long long grid = sms;  // one CTA (4 DMMA warps + 1 producer) per SM
  if (grid > total) grid = total;
  zgemm_dmma_ws<A_MK, B_KN><<<(unsigned)grid, NT3, Cfg::SMEM, st>>>(*b, total);
  return cudaGetLastError();
}

}  // namespace

int gemm_variant() {
  // MICCO_GEMM = 1 per-tile 64×64, 2 persistent 64×64 4M, 3 warp-specialized, 5 persistent 64×32 3M
  // (default: 19.7k vs 18.8k graphs/s for 2 on the bench workload, profiles/bench_r01_v4.json),
  // 6 small 32×32 (4 stages, 3 CTAs/SM), 7 64×32, 8 32×32 (3 stages, 4 CTAs/SM)
  static int variant = -1;
  if (variant < 0) {
    const char *e = getenv("MICCO_GEMM");
    variant = (e && e[0] >= '1' && e[0] <= '8') ? e[0] - '0' : 5;
  }
  return variant;
}

void gemm_tile_shape(int cls, int *bm, int *bn) {
  const int v = gemm_variant();
  *bm = 64;
  *bn = 64;
  if (cls == 4) return;  // gather kernel (v1)
  if (v == 6 || v == 8) { *bm = 32; *bn = 32; }
  if (v == 7 || v == 5) { *bm = 64; *bn = 32; }
}

bool gemm_uses_3m(int cls) { return cls != 4 && (gemm_variant() == 5 || gemm_variant() == 4); }

cudaError_t launch_gemm_group(const GemmBatch *b, long long total_tiles, int cls, cudaStream_t st) {
  static bool attr_set = false;  // per process; the attribute is per-function, all devices
  const int variant = gemm_variant();
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(zgemm_dmma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, GEMM_SMEM);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(zgemm_persistent<2, 2, 32, 32, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             PCfg<64, 64>::SMEM);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(zgemm_persistent<2, 2, 32, 16, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             PCfg<64, 32>::SMEM);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  if (total_tiles <= 0) return cudaSuccess;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (variant == 1 || cls == 4) {
    long long grid = total_tiles < (1LL << 30) ? total_tiles : (1LL << 30);
    zgemm_dmma_kernel<<<(unsigned)grid, NT, GEMM_SMEM, st>>>(*b, total_tiles);
    return cudaGetLastError();
  }
  if (variant == 6 || variant == 7 || variant == 8) {
    // tile sizes must match the host's tilesM/tilesN (kGemmBM/BN for the other variants)
    long long grid = total_tiles;
    if (variant == 6) {
      using C6 = SmallCfg<32, 32, 4>;
      static bool a6 = false;
      if (!a6) { cudaFuncSetAttribute(zgemm_small<32, 32, 4, 3>, cudaFuncAttributeMaxDynamicSharedMemorySize, C6::SMEM); a6 = true; }
      zgemm_small<32, 32, 4, 3><<<(unsigned)grid, 128, C6::SMEM, st>>>(*b, total_tiles);
    } else if (variant == 7) {
      using C7 = SmallCfg<64, 32, 4>;
      static bool a7 = false;
      if (!a7) { cudaFuncSetAttribute(zgemm_small<64, 32, 4, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, C7::SMEM); a7 = true; }
      zgemm_small<64, 32, 4, 2><<<(unsigned)grid, 128, C7::SMEM, st>>>(*b, total_tiles);
    } else {
      using C8 = SmallCfg<32, 32, 3>;
      static bool a8 = false;
      if (!a8) { cudaFuncSetAttribute(zgemm_small<32, 32, 3, 4>, cudaFuncAttributeMaxDynamicSharedMemorySize, C8::SMEM); a8 = true; }
      zgemm_small<32, 32, 3, 4><<<(unsigned)grid, 128, C8::SMEM, st>>>(*b, total_tiles);
    }
    return cudaGetLastError();
  }
  if (variant == 4) {  // 3M, 8 warps of 32×16 on a 64×64 tile, one CTA per SM (255 registers)
    static bool a4 = false;
    if (!a4) {
      cudaFuncSetAttribute(zgemm_persistent1<2, 4, 32, 16, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           PCfg<64, 64>::SMEM);
      a4 = true;
    }
    long long grid = sms;
    if (grid > total_tiles) grid = total_tiles;
    zgemm_persistent1<2, 4, 32, 16, true><<<(unsigned)grid, 256, PCfg<64, 64>::SMEM, st>>>(*b, total_tiles);
    return cudaGetLastError();
  }
  if (variant == 2 || variant == 5) {
    long long grid = 2LL * sms;  // 2 resident CTAs per SM (112 KB smem each)
    if (grid > total_tiles) grid = total_tiles;
    if (variant == 2)
      zgemm_persistent<2, 2, 32, 32, false><<<(unsigned)grid, 128, PCfg<64, 64>::SMEM, st>>>(*b, total_tiles);
    else  // 5: 3M complex products, 64×32 CTA tile
      zgemm_persistent<2, 2, 32, 16, true><<<(unsigned)grid, 128, PCfg<64, 32>::SMEM, st>>>(*b, total_tiles);
    return cudaGetLastError();
  }
  switch (cls) {
    case 0: return launch_ws<true, true>(b, total_tiles, sms, st);
    case 1: return launch_ws<true, false>(b, total_tiles, sms, st);
    case 2: return launch_ws<false, true>(b, total_tiles, sms, st);
    default: return launch_ws<false, false>(b, total_tiles, sms, st);
  }
}

cudaError_t launch_dot_group(const DotBatch *b, long long total_ctas, cudaStream_t st) {
  if (total_ctas <= 0) return cudaSuccess;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(zdot_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, DOT_SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  zdot_kernel<<<(unsigned)total_ctas, DT, DOT_SMEM, st>>>(*b);
  return cudaGetLastError();
}

cudaError_t launch_finalize(int G, int Lt, const int *comp_off, const int *comp_slot, const double2 *scalars,
                            double2 *vals, cudaStream_t st) {
  long long n = (long long)G * Lt;
  if (n == 0) return cudaSuccess;
  finalize_kernel<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(G, Lt, comp_off, comp_slot, scalars, vals);
  return cudaGetLastError();
}

cudaError_t launch_correlator_sum(int G, int Lt, const double2 *coefs, const double2 *vals, double2 *corr,
                                  cudaStream_t st) {
  corr_sum_kernel<<<Lt, DT, 0, st>>>(G, Lt, coefs, vals, corr);
  return cudaGetLastError();
}

cudaError_t launch_accumulate(double2 *dst, const double2 *src, long long n, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  long long blocks = (n + 255) / 256;
  if (blocks > 148 * 16) blocks = 148 * 16;
  accumulate_kernel<<<(unsigned)blocks, 256, 0, st>>>(dst, src, n);
  return cudaGetLastError();
}

}  // namespace micco
