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
#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include <cudaTypedefs.h>

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
__device__ __forceinline__ void cp_async16s(unsigned s, const void *gmem, bool valid) {
  int sz = valid ? 16 : 0;
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(s), "l"(gmem), "r"(sz));
}
__device__ __forceinline__ void cp_async16s(unsigned s, const void *gmem) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem));
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

// ---------------------------------------------------------------- persistent GEMM (v2, 3M)
//
// The production GEMM.  Persistent CTAs (2 per SM) take every G-th tile and run one
// continuous cp.async pipeline (BK = 16, 3 stages) over their whole (tile, k-step) sequence;
// the next stage's copies are issued in NPART pieces inside the DMMA stream of the stage being
// computed so they occupy the DMMA pacing slots; the task descriptor advances linearly.
// Optional fused final dot (GemmDesc::D) in the epilogue.
//
// Complex product: the 3M "T" (Gauss) form, T1 += Ar·Br, T2 += Ai·Bi, T3 += (Ar+Ai)·(Br+Bi);
// Cr = T1 − T2, Ci = T3 − (T1 + T2): 3 DMMAs per 8×8×4 complex block instead of the textbook
// 4, for the same algorithmic work (8 real flops per complex MAC are still what the roofline
// counts).  Its rounding differs from the 4M form but stays far inside the 1e-10 parity bound,
// and exact-integer inputs stay bit-exact (every partial sum is an integer below 2^53; SURVEY.md
// §8(c) "Bit-exact GPU parity").  The operand sums are DADDs on the FP64 pipe the DMMAs occupy;
// the T form needs MI + NJ of them per k-quad (the "K" form K1 = (Ar+Ai)·Br, K2 = Ar·(Bi−Br),
// K3 = Ai·(Br+Bi) needs MI + 2·NJ and ran at 35.0 instead of 36.9 TFLOP/s; the 4M kernel at
// 31.6; measured round 1).
constexpr int BK2 = 16, ST2 = 3;
constexpr int APITCH2 = BK2 + 4;  // [m][k] rows: 320 B ≡ 64 (mod 128): A fragment loads conflict-free

template <int TBM, int TBN>
struct PCfg {
  static constexpr int BP = TBN + 2;  // [k][n] rows: (TBN+2)·16 B ≡ 32 (mod 128) for TBN ∈ {32, 64}
  static constexpr int AE = TBM * APITCH2, BE = BK2 * BP;
  static constexpr int SMEM = ST2 * (AE + BE) * 16;
};

// Per-thread load geometry of one operand stage, compile-time for a layout class.  A stage
// holds ROWS × BK2 complex elements (rows = m for A, n for B); KFAST = the operand is
// contiguous along k, so consecutive threads copy consecutive k.  Element j of a thread sits
// at (row r0 + j·RJ, k k0 + j·KJ): its shared-memory offset advances by a compile-time
// stride and its global offset by a per-tile constant, so a copy is one IMAD.WIDE + LDGSTS.
template <int ROWS, int NTH, bool KFAST>
struct Geo {
  static constexpr int L = ROWS * BK2 / NTH;
  static constexpr int RJ = KFAST ? NTH / BK2 : 0;
  static constexpr int KJ = KFAST ? 0 : NTH / ROWS;
  static_assert(KFAST ? (NTH % BK2 == 0) : (NTH % ROWS == 0), "load geometry");
  __device__ static int r0(int tid) { return KFAST ? tid / BK2 : tid % ROWS; }
  __device__ static int k0(int tid) { return KFAST ? tid % BK2 : tid / ROWS; }
};

// bits j < L with base + j·STEP < lim
template <int L, int STEP>
__device__ __forceinline__ unsigned run_mask(int base, int lim) {
  const int room = lim - base;
  if (room <= 0) return 0u;
  if constexpr (STEP == 0) {
    return (1u << L) - 1u;
  } else {
    const int cnt = min(L, (room + STEP - 1) / STEP);
    return (1u << cnt) - 1u;
  }
}

template <int LA, int LB>
struct LoadCur {
  static constexpr int NA = LA, NB = LB;
  const double2 *A, *B;    // tile bases (t, mo/no, m0/n0 applied; ko = kb = 0)
  const double2 *pA, *pB;  // bases of the stage being loaded
  long long sAko, sBko;
  int stepA, stepB;        // BK2·sAki, BK2·sBki
  int Ki, KT, KTOT, kin, ko, kb;
  int gA[LA], gB[LB];      // element offsets from the stage base (0 for rows outside the tile)
  unsigned rmA, rmB;       // rows inside the tile
  // blocked-K geometry (class kGemmClassKB): a stage is 4 ko × 4 ki, local k = 4·dko + dki;
  // element j of a thread has local k kl0 + j·kls, shared offset s0 + j·sj (bytes)
  int sAki, sBki, Ko, ko0, ki0;
  int klA0, klAs, klB0, klBs;
  unsigned sa0, sb0, sja, sjb;
};

// Per-thread blocked-K geometry of one operand (rows = m for A, n for B): the copy order
// follows the operand's unit-stride index (ko, ki or the row), so warps read 64-byte runs.
template <int ROWS, int NTH>
__device__ __forceinline__ void kb_geo(int tid, long long sRow, long long sKo, long long sKi, int &r0, int &rj,
                                       int &kl0, int &kls) {
  if (sRow == 1 && sKo != 1 && sKi != 1) {  // row-fast
    r0 = tid % ROWS; rj = 0; kl0 = tid / ROWS; kls = NTH / ROWS;
  } else if (sKo == 1) {                     // ko-fast: dko = tid & 3, dki = (tid >> 2) & 3
    r0 = tid / BK2; rj = NTH / BK2; kl0 = (tid & 3) * 4 + ((tid >> 2) & 3); kls = 0;
  } else {                                   // ki-fast (also the gather fallback)
    r0 = tid / BK2; rj = NTH / BK2; kl0 = tid & (BK2 - 1); kls = 0;
  }
}

struct StoreCur {
  double2 *C;
  int sCmi, sCni, Mi, Ni, m0, n0, KTOT;
  const double2 *D;  // fused final dot: the partner tile base (nullptr = plain GEMM)
  long long pidx;    // first partial-sum slot of this tile
};

template <int NTH, int TBM, int TBN, bool AKF, bool BNF, bool KB, typename LC>
__device__ __forceinline__ void decode_tile(const GemmDesc *__restrict__ descs, int n_desc, int &task,
                                            long long tile, int tid, LC *L, StoreCur *S) {
  using GA = Geo<TBM, NTH, AKF>;
  using GB = Geo<TBN, NTH, !BNF>;
  while (task + 1 < n_desc && descs[task + 1].tile_begin <= tile) ++task;
  const GemmDesc &d = descs[task];
  unsigned lt = (unsigned)(tile - d.tile_begin);  // tiles of one task < 2^32: 32-bit div/mod
  const unsigned tilesN = d.tilesN, tilesM = d.tilesM, No = d.No, Mo = d.Mo;
  const int tn = (int)(lt % tilesN); lt /= tilesN;
  const int tm = (int)(lt % tilesM); lt /= tilesM;
  const int no = (int)(lt % No); lt /= No;
  const int mo = (int)(lt % Mo);
  const long long t = lt / Mo;
  const int m0 = tm * TBM, n0 = tn * TBN;
  const int KT = KB ? ((d.Ko + 3) / 4) * ((d.Ki + 3) / 4) : (d.Ki + BK2 - 1) / BK2;
  if (KB && L) {
    const int sAmi = (int)d.sAmi, sBni = (int)d.sBni;
    L->A = d.A + t * d.sAt + mo * d.sAmo + (long long)m0 * sAmi;
    L->B = d.B + t * d.sBt + no * d.sBno + (long long)n0 * sBni;
    L->pA = L->A; L->pB = L->B;
    L->sAko = d.sAko; L->sBko = d.sBko;
    L->sAki = (int)d.sAki; L->sBki = (int)d.sBki;
    L->Ki = d.Ki; L->Ko = d.Ko; L->KT = KT; L->KTOT = KT;
    L->ko0 = 0; L->ki0 = 0;
    int ra, rja, rb, rjb;
    kb_geo<TBM, NTH>(tid, d.sAmi, d.sAko, d.sAki, ra, rja, L->klA0, L->klAs);
    kb_geo<TBN, NTH>(tid, d.sBni, d.sBko, d.sBki, rb, rjb, L->klB0, L->klBs);
    L->sa0 = (unsigned)((ra * APITCH2 + L->klA0) * 16);
    L->sja = (unsigned)((rja * APITCH2 + L->klAs) * 16);
    L->sb0 = (unsigned)((L->klB0 * PCfg<TBM, TBN>::BP + rb) * 16);
    L->sjb = (unsigned)((L->klBs * PCfg<TBM, TBN>::BP + rjb) * 16);
    L->rmA = L->rmB = 0;
#pragma unroll
    for (int j = 0; j < LC::NA; ++j) {
      const int m = ra + j * rja, kl = L->klA0 + j * L->klAs;
      const bool v = m0 + m < d.Mi;
      if (v) L->rmA |= 1u << j;
      L->gA[j] = v ? (int)(m * d.sAmi + (kl >> 2) * d.sAko + (kl & 3) * d.sAki) : 0;
    }
#pragma unroll
    for (int j = 0; j < LC::NB; ++j) {
      const int n = rb + j * rjb, kl = L->klB0 + j * L->klBs;
      const bool v = n0 + n < d.Ni;
      if (v) L->rmB |= 1u << j;
      L->gB[j] = v ? (int)(n * d.sBni + (kl >> 2) * d.sBko + (kl & 3) * d.sBki) : 0;
    }
  } else if (L) {
    const int sAmi = (int)d.sAmi, sAki = (int)d.sAki, sBki = (int)d.sBki, sBni = (int)d.sBni;
    L->A = d.A + t * d.sAt + mo * d.sAmo + (long long)m0 * sAmi;
    L->B = d.B + t * d.sBt + no * d.sBno + (long long)n0 * sBni;
    L->pA = L->A; L->pB = L->B;
    L->sAko = d.sAko; L->sBko = d.sBko;
    L->stepA = BK2 * sAki; L->stepB = BK2 * sBki;
    L->Ki = d.Ki; L->KT = KT; L->KTOT = d.Ko * KT;
    L->kin = 0; L->ko = 0; L->kb = 0;
    const int ra = GA::r0(tid), ka = GA::k0(tid), rb = GB::r0(tid), kb = GB::k0(tid);
    L->rmA = run_mask<GA::L, GA::RJ>(m0 + ra, d.Mi);
    L->rmB = run_mask<GB::L, GB::RJ>(n0 + rb, d.Ni);
    const int bA = ra * sAmi + ka * sAki, jA = GA::RJ * sAmi + GA::KJ * sAki;
    const int bB = kb * sBki + rb * sBni, jB = GB::KJ * sBki + GB::RJ * sBni;
#pragma unroll
    for (int j = 0; j < GA::L; ++j) L->gA[j] = ((L->rmA >> j) & 1u) ? bA + j * jA : 0;
#pragma unroll
    for (int j = 0; j < GB::L; ++j) L->gB[j] = ((L->rmB >> j) & 1u) ? bB + j * jB : 0;
  }
  if (S) {
    S->C = d.C + t * d.sCt + mo * d.sCmo + no * d.sCno;
    S->sCmi = (int)d.sCmi; S->sCni = (int)d.sCni;
    S->Mi = d.Mi; S->Ni = d.Ni; S->m0 = m0; S->n0 = n0;
    S->KTOT = KB ? KT : d.Ko * KT;
    S->D = d.D ? d.D + t * d.sDt + mo * d.sDmo + no * d.sDno : nullptr;
    S->pidx = (tile - d.tile_begin) * (NTH / 32);
  }
}

// NWM × NWN warps with WTM × WTN complex warp tiles; CTA tile (NWM·WTM) × (NWN·WTN).
// AKF / BNF: the layout class (A contiguous along k / B contiguous along n).
template <int NWM, int NWN, int WTM, int WTN, bool AKF, bool BNF, bool KB = false>
__device__ __forceinline__ void zgemm_persistent_body(const GemmDesc *__restrict__ descs, int n_desc,
                                                      long long total) {
  constexpr int NTH = NWM * NWN * 32;
  constexpr int TBM = NWM * WTM, TBN = NWN * WTN;
  using GA = Geo<TBM, NTH, AKF>;  // (KB: only the element counts are used)
  using GB = Geo<TBN, NTH, !BNF>;
  constexpr int LPTA = GA::L, LPTB = GB::L;
  constexpr int MI = WTM / 8, NJ = WTN / 8;  // 8x8 blocks per warp
  constexpr int NACC = 3;  // T1, T2, T3
  using Cfg = PCfg<TBM, TBN>;
  constexpr int BP = Cfg::BP;
  // shared-memory stride between a thread's consecutive elements (complex elements)
  constexpr int SJA = GA::RJ * APITCH2 + GA::KJ, SJB = GB::KJ * BP + GB::RJ;
  extern __shared__ __align__(128) double2 smem[];
  double2 *As = smem;
  double2 *Bs = smem + ST2 * Cfg::AE;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int wm = warp / NWN, wn = warp % NWN;
  const unsigned sA0 = (unsigned)__cvta_generic_to_shared(As + GA::r0(tid) * APITCH2 + GA::k0(tid));
  const unsigned sB0 = (unsigned)__cvta_generic_to_shared(Bs + GB::k0(tid) * BP + GB::r0(tid));
  const unsigned sAs = (unsigned)__cvta_generic_to_shared(As), sBs = (unsigned)__cvta_generic_to_shared(Bs);

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
  decode_tile<NTH, TBM, TBN, AKF, BNF, KB>(descs, n_desc, task_l, tile_l, tid, &L, &S);
  // The load side decodes every tile first; it leaves the store cursor of that tile in Sn so
  // the epilogue does not decode it again (unless the loads ran more than a tile ahead).
  StoreCur Sn;
  long long sn_tile = -1;
  int sn_task = 0;
  bool more_l = true;

  // The loads of a stage are issued in NPART pieces interleaved with the DMMA stream of the
  // stage being computed (one piece per k-quad), so the scheduler can slot the cp.async
  // into the DMMA pacing gaps instead of running a separate load phase.  A DMMA holds its
  // warp for 15 cycles (its SASS stall count), so with two warps per scheduler each has
  // ~16 free issue cycles per DMMA: the copies must cost a few instructions, not dozens.
  constexpr int NPART = BK2 / 4;
  static_assert(LPTA % NPART == 0 && LPTB % NPART == 0, "load split");
  unsigned mA = 0, mB = 0;  // elements of the stage being loaded inside the operand
  bool ld_full = false;     // ... all of them (interior tile, whole k-step): warp-uniform
  auto begin_load = [&]() {
    if constexpr (KB) {
      if (L.ko0 + 4 <= L.Ko && L.ki0 + 4 <= L.Ki) {
        mA = L.rmA;
        mB = L.rmB;
      } else {
        unsigned ka = 0, kb = 0;
#pragma unroll
        for (int j = 0; j < LPTA; ++j) {
          const int kl = L.klA0 + j * L.klAs;
          if (L.ko0 + (kl >> 2) < L.Ko && L.ki0 + (kl & 3) < L.Ki) ka |= 1u << j;
        }
#pragma unroll
        for (int j = 0; j < LPTB; ++j) {
          const int kl = L.klB0 + j * L.klBs;
          if (L.ko0 + (kl >> 2) < L.Ko && L.ki0 + (kl & 3) < L.Ki) kb |= 1u << j;
        }
        mA = L.rmA & ka;
        mB = L.rmB & kb;
      }
    } else {
      mA = L.rmA & run_mask<LPTA, GA::KJ>(L.kb + GA::k0(tid), L.Ki);
      mB = L.rmB & run_mask<LPTB, GB::KJ>(L.kb + GB::k0(tid), L.Ki);
    }
    if constexpr (!KB) ld_full = __all_sync(0xffffffffu, mA == (1u << LPTA) - 1u && mB == (1u << LPTB) - 1u);
  };
  auto issue_part = [&](int slot, int part) {
    if constexpr (KB) {  // runtime geometry (per task): element j at s0 + j·sj
      const unsigned sa = sAs + slot * (Cfg::AE * 16) + L.sa0, sb = sBs + slot * (Cfg::BE * 16) + L.sb0;
#pragma unroll
      for (int jj = 0; jj < LPTA / NPART; ++jj) {
        const int j = part * (LPTA / NPART) + jj;
        const bool v = (mA >> j) & 1u;
        cp_async16s(sa + j * L.sja, L.pA + (v ? L.gA[j] : 0), v);
      }
#pragma unroll
      for (int jj = 0; jj < LPTB / NPART; ++jj) {
        const int j = part * (LPTB / NPART) + jj;
        const bool v = (mB >> j) & 1u;
        cp_async16s(sb + j * L.sjb, L.pB + (v ? L.gB[j] : 0), v);
      }
      return;
    }
    const unsigned sa = sA0 + slot * (Cfg::AE * 16), sb = sB0 + slot * (Cfg::BE * 16);
    if (ld_full) {  // every element inside both operands: plain copies, no zero fill
#pragma unroll
      for (int jj = 0; jj < LPTA / NPART; ++jj) {
        const int j = part * (LPTA / NPART) + jj;
        cp_async16s(sa + j * SJA * 16, L.pA + L.gA[j]);
      }
#pragma unroll
      for (int jj = 0; jj < LPTB / NPART; ++jj) {
        const int j = part * (LPTB / NPART) + jj;
        cp_async16s(sb + j * SJB * 16, L.pB + L.gB[j]);
      }
      return;
    }
#pragma unroll
    for (int jj = 0; jj < LPTA / NPART; ++jj) {
      const int j = part * (LPTA / NPART) + jj;
      const bool v = (mA >> j) & 1u;
      cp_async16s(sa + j * SJA * 16, L.pA + (v ? L.gA[j] : 0), v);
    }
#pragma unroll
    for (int jj = 0; jj < LPTB / NPART; ++jj) {
      const int j = part * (LPTB / NPART) + jj;
      const bool v = (mB >> j) & 1u;
      cp_async16s(sb + j * SJB * 16, L.pB + (v ? L.gB[j] : 0), v);
    }
  };
  auto advance_load = [&]() {  // next k-step, possibly in the next tile
    if (++kt_l == L.KTOT) {
      kt_l = 0;
      if ((tile_l += G) < total) {
        decode_tile<NTH, TBM, TBN, AKF, BNF, KB>(descs, n_desc, task_l, tile_l, tid, &L, &Sn);
        sn_tile = tile_l;
        sn_task = task_l;
      } else {
        more_l = false;
      }
    } else if constexpr (KB) {
      if ((L.ki0 += 4) >= L.Ki) {
        L.ki0 = 0;
        L.ko0 += 4;
      }
      L.pA = L.A + L.ko0 * L.sAko + L.ki0 * L.sAki;
      L.pB = L.B + L.ko0 * L.sBko + L.ki0 * L.sBki;
    } else if (++L.kin == L.KT) {
      L.kin = 0; L.kb = 0; ++L.ko;
      L.pA = L.A + L.ko * L.sAko;
      L.pB = L.B + L.ko * L.sBko;
    } else {
      L.kb += BK2;
      L.pA += L.stepA;
      L.pB += L.stepB;
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
  // Fragments are double-buffered: the LDS and the operand sums of k-quad q+1 are issued
  // before the DMMAs of q.  (The stage barrier sits at the top of the stage: moving it before
  // the DMMAs of the last k-quad measured slower, 35.6 vs 36.9 TF, round 1.)
  double fa[2][MI][3], fb[2][NJ][3];
  auto load_frag = [&](int buf, int slot, int kq) {
    const double2 *as = As + slot * Cfg::AE;
    const double2 *bs = Bs + slot * Cfg::BE;
#pragma unroll
    for (int i = 0; i < MI; ++i) {
      const double2 a = as[(wm * WTM + i * 8 + (lane >> 2)) * APITCH2 + kq * 4 + (lane & 3)];
      fa[buf][i][0] = a.x;
      fa[buf][i][1] = a.y;
      fa[buf][i][2] = a.x + a.y;  // Ar + Ai
    }
#pragma unroll
    for (int j = 0; j < NJ; ++j) {
      const double2 b = bs[(kq * 4 + (lane & 3)) * BP + wn * WTN + j * 8 + (lane >> 2)];
      fb[buf][j][0] = b.x;
      fb[buf][j][1] = b.y;
      fb[buf][j][2] = b.x + b.y;  // Br + Bi
    }
  };
  for (;;) {
    cp_async_wait<ST2 - 2>();
    __syncthreads();
    load_frag(0, slot_c, 0);
    const bool ld = more_l;
    if (ld) begin_load();
#pragma unroll
    for (int kq = 0; kq < BK2 / 4; ++kq) {
      if (ld) issue_part(slot_l, kq);
      const int cur = kq & 1;
      if (kq + 1 < BK2 / 4) {
        load_frag(cur ^ 1, slot_c, kq + 1);
      } else {
        if (ld) advance_load();
        cp_async_commit();
      }
#pragma unroll
      for (int i = 0; i < MI; ++i)
#pragma unroll
        for (int j = 0; j < NJ; ++j) {
          dmma(acc[i][j][0][0], acc[i][j][0][1], fa[cur][i][0], fb[cur][j][0]);  // Ar·Br
          dmma(acc[i][j][1][0], acc[i][j][1][1], fa[cur][i][1], fb[cur][j][1]);  // Ai·Bi
          dmma(acc[i][j][2][0], acc[i][j][2][1], fa[cur][i][2], fb[cur][j][2]);  // (Ar+Ai)·(Br+Bi)
        }
    }
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
      auto cval = [&](int i, int j, int h, double &re, double &im) {  // T1 − T2, T3 − (T1 + T2)
        re = acc[i][j][0][h] - acc[i][j][1][h];
        im = acc[i][j][2][h] - (acc[i][j][0][h] + acc[i][j][1][h]);
      };
      if (S.D) {
        // fused final contraction: this warp's partial Σ C·D (no C written)
        const GemmDesc &dd = descs[task_c];
        const long long sDmi = dd.sDmi, sDni = dd.sDni;
        // partner loads: all rows issued before their use (one round trip to L2, where the
        // block was prefetched)
        constexpr int CH = MI;
        double pr = 0.0, pim = 0.0;
#pragma unroll
        for (int i0 = 0; i0 < MI; i0 += CH) {
          double2 y[CH][NJ][2];
#pragma unroll
          for (int ii = 0; ii < CH; ++ii) {
            const int m = S.m0 + wm * WTM + (i0 + ii) * 8 + (lane >> 2);
#pragma unroll
            for (int j = 0; j < NJ; ++j)
#pragma unroll
              for (int h = 0; h < 2; ++h) {
                const int n = S.n0 + wn * WTN + j * 8 + (lane & 3) * 2 + h;
                y[ii][j][h] = (m < S.Mi && n < S.Ni) ? S.D[(long long)m * sDmi + (long long)n * sDni]
                                                     : make_double2(0.0, 0.0);
              }
          }
#pragma unroll
          for (int ii = 0; ii < CH; ++ii)
#pragma unroll
            for (int j = 0; j < NJ; ++j)
#pragma unroll
              for (int h = 0; h < 2; ++h) {
                double re, im;
                cval(i0 + ii, j, h, re, im);
                pr += re * y[ii][j][h].x - im * y[ii][j][h].y;
                pim += re * y[ii][j][h].y + im * y[ii][j][h].x;
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
      if (sn_tile == tile_c) {
        S = Sn;
        task_c = sn_task;
      } else {
        decode_tile<NTH, TBM, TBN, AKF, BNF, KB>(descs, n_desc, task_c, tile_c, tid, (LoadCur<LPTA, LPTB> *)nullptr, &S);
      }
    }
  }
  cp_async_wait<0>();
}

// ---------------------------------------------------------------- TMA warp-specialized GEMM (3M)
//
// The production GEMM for contractions whose operands fit 5-D tensor maps (every meson GEMM;
// gemm_tma_class).  One CTA per SM: two consumer warpgroups (8 warps, 4 × 2, warp tile 32 × 16
// complex, 3M "T" accumulators; CTA tile 128 × 32) and one producer warpgroup whose elected lane
// streams the operand stages with TMA (cp.async.bulk.tensor, SASS UTMALDG) through a 5-slot
// shared-memory ring guarded by full/empty mbarriers.  Registers are allocated per warpgroup
// (a 9-warp CTA is charged for 12): the kernel launches at 168 per thread, then the producer
// warpgroup gives back to 40 and the consumers grow to 232 (setmaxnreg).  The consumers' loop is fragment LDS + operand-sum DADD + DMMA plus one
// mbarrier wait and one arrive per stage: no per-thread copy addressing, no bounds masks (TMA
// zero-fills ragged tiles) and no CTA-wide barrier (the cp.async kernel above spent ~180
// non-DMMA instructions per 96 DMMAs per stage on them, ncu profiles/ncu_gemm_c3_r02.json).
//
// The tensor maps lay each stage out for conflict-free 16-byte fragment loads without padding
// (probe: tools/tma_probe.cu):
//   K-major operand (contiguous along k):   smem [kq][row][k4]      (lane (r, c) of an 8-row
//                                           block reads 32 consecutive complex)
//   MN-major operand (contiguous along row): smem [kq][row/2][k4][2] (lanes 0-7 = rows 0-1 ×
//                                           k 0-3 hit 8 distinct 16-byte bank groups)
// where kq = k / 4 and k4 = k % 4: the map's dimensions step through the operand in that order
// (non-monotonic global strides, accepted by cuTensorMapEncodeTiled).
constexpr int TM_NWM = 4, TM_NWN = 2, TM_NW = TM_NWM * TM_NWN;  // consumer warps
constexpr int TM_BM = TM_NWM * 32, TM_BN = TM_NWN * 16, TM_BK = 16, TM_ST = 5;
constexpr int TM_THREADS = (TM_NW + 4) * 32;  // + the producer warpgroup
constexpr int TM_REG_LAUNCH = 168, TM_REG_PRODUCER = 40, TM_REG_CONSUMER = 232;
static_assert(TM_THREADS * TM_REG_LAUNCH <= 65536, "register file");
static_assert(4 * 32 * (TM_REG_LAUNCH - TM_REG_PRODUCER) >= TM_NW * 32 * (TM_REG_CONSUMER - TM_REG_LAUNCH),
              "setmaxnreg balance");
constexpr int TM_AE = TM_BM * TM_BK, TM_BE = TM_BN * TM_BK;  // complex per stage
constexpr int TM_STAGE_BYTES = (TM_AE + TM_BE) * 16;
constexpr int TM_SMEM = TM_ST * TM_STAGE_BYTES + 2 * TM_ST * 8;

__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned bar, unsigned cnt) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(cnt) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned bar, unsigned parity) {
  asm volatile(
      "{\n .reg .pred p;\n TMW_%=: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra TMW_%=;\n}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load5(unsigned dst, const CUtensorMap *m, unsigned bar, int c0, int c1, int c2, int c3,
                                          int c4) {
  asm volatile(
      "cp.async.bulk.tensor.5d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(
          dst),
      "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4), "r"(bar)
      : "memory");
}

// tile → (task, t, mo, no, m0, n0); descriptors advance linearly (tiles increase)
struct TmTile {
  int t, mo, no, m0, n0;
};
__device__ __forceinline__ TmTile tm_decode(const GemmDesc *__restrict__ descs, int n_desc, int &task, long long tile) {
  while (task + 1 < n_desc && descs[task + 1].tile_begin <= tile) ++task;
  const GemmDesc &d = descs[task];
  unsigned lt = (unsigned)(tile - d.tile_begin);  // < 2^32 tiles per task (executor.cu check)
  TmTile r;
  const unsigned tilesN = d.tilesN, tilesM = d.tilesM, No = d.No, Mo = d.Mo;
  const int tn = (int)(lt % tilesN); lt /= tilesN;
  const int tm = (int)(lt % tilesM); lt /= tilesM;
  r.no = (int)(lt % No); lt /= No;
  r.mo = (int)(lt % Mo);
  r.t = (int)(lt / Mo);
  r.m0 = tm * TM_BM;
  r.n0 = tn * TM_BN;
  return r;
}

// Fragment offset (complex) of lane within an 8-row block, per operand layout.
template <bool KMAJ>
__device__ __forceinline__ int tm_lane_off(int lane) {
  if constexpr (KMAJ) return lane;                        // row·4 + k4
  const int r = lane >> 2, c = lane & 3;
  return (r >> 1) * 8 + c * 2 + (r & 1);                 // (row/2)·8 + k4·2 + row%2
}

template <bool AK, bool BK>
__device__ __forceinline__ void zgemm_tma_body(const GemmTmaBatch &b, long long total) {
  constexpr int MI = 4, NJ = 2;  // 8×8 blocks per warp (32 × 16 complex)
  extern __shared__ __align__(128) double2 smem[];
  double2 *As = smem;                    // [TM_ST][TM_AE]
  double2 *Bs = smem + TM_ST * TM_AE;    // [TM_ST][TM_BE]
  unsigned long long *bars = reinterpret_cast<unsigned long long *>(Bs + TM_ST * TM_BE);
  const unsigned full0 = smem_u32(bars), empty0 = smem_u32(bars + TM_ST);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const GemmDesc *__restrict__ descs = b.d;
  const int n_desc = b.n;
  const long long G = gridDim.x;
  if (tid == 0) {
    for (int i = 0; i < TM_ST; ++i) {
      mbar_init(full0 + 8 * i, 1);   // the producer's arrive.expect_tx (+ the TMA bytes)
      mbar_init(empty0 + 8 * i, TM_NW);  // one arrive per consumer warp
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if ((long long)blockIdx.x >= total) return;
  int task0 = 0;
  {
    int lo = 0, hi = n_desc - 1;
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (descs[mid].tile_begin <= (long long)blockIdx.x) lo = mid; else hi = mid - 1;
    }
    task0 = lo;
  }

  if (warp >= TM_NW) {  // ---------------- producer warpgroup: one lane streams every stage
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(TM_REG_PRODUCER));
    if (warp != TM_NW || lane != 0) return;
    int task = task0, slot = 0;
    unsigned ph = 0;
    int prefetched = -1;
    for (long long tile = blockIdx.x; tile < total; tile += G) {
      const TmTile tt = tm_decode(descs, n_desc, task, tile);
      const GemmDesc &d = descs[task];
      const CUtensorMap *ma = &b.map[2 * task], *mb = &b.map[2 * task + 1];
      if (task != prefetched) {
        asm volatile("prefetch.tensormap [%0];" ::"l"(ma) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(mb) : "memory");
        prefetched = task;
      }
      const int kti = (d.Ki + TM_BK - 1) / TM_BK;
      const int ks_n = d.Ko * kti;
      for (int ks = 0; ks < ks_n; ++ks) {
        const int ko = ks / kti, kq0 = (ks - ko * kti) * (TM_BK / 4);
        mbar_wait(empty0 + 8 * slot, ph ^ 1);
        const unsigned fb = full0 + 8 * slot;
        mbar_expect_tx(fb, TM_STAGE_BYTES);
        const unsigned sa = smem_u32(As + slot * TM_AE), sb = smem_u32(Bs + slot * TM_BE);
        if constexpr (AK) tma_load5(sa, ma, fb, 0, tt.m0, kq0, tt.t, d.Ko > 1 ? ko : tt.mo);
        else tma_load5(sa, ma, fb, 0, 0, tt.m0 >> 1, kq0, tt.t);
        if constexpr (BK) tma_load5(sb, mb, fb, 0, tt.n0, kq0, tt.t, d.Ko > 1 ? ko : tt.no);
        else tma_load5(sb, mb, fb, 0, 0, tt.n0 >> 1, kq0, tt.t);
        if (++slot == TM_ST) { slot = 0; ph ^= 1; }
      }
    }
    return;
  }

  // ---------------- consumers: TM_NWM × TM_NWN warps
  asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(TM_REG_CONSUMER));
  const int wm = warp / TM_NWN, wn = warp % TM_NWN;
  const int aoff = wm * 128 + tm_lane_off<AK>(lane);  // + kq·(TM_BM·4) + i·32
  const int boff = wn * 64 + tm_lane_off<BK>(lane);   // + kq·(TM_BN·4) + j·32
  double acc[MI][NJ][3][2];
#pragma unroll
  for (int i = 0; i < MI; ++i)
#pragma unroll
    for (int j = 0; j < NJ; ++j)
#pragma unroll
      for (int q = 0; q < 3; ++q) acc[i][j][q][0] = acc[i][j][q][1] = 0.0;
  double fa[2][MI][3], fb[2][NJ][3];
  auto load_frag = [&](int buf, int slot, int kq) {
    const double2 *as = As + slot * TM_AE + kq * (TM_BM * 4) + aoff;
    const double2 *bs = Bs + slot * TM_BE + kq * (TM_BN * 4) + boff;
#pragma unroll
    for (int i = 0; i < MI; ++i) {
      const double2 a = as[i * 32];
      fa[buf][i][0] = a.x;
      fa[buf][i][1] = a.y;
      fa[buf][i][2] = a.x + a.y;  // Ar + Ai
    }
#pragma unroll
    for (int j = 0; j < NJ; ++j) {
      const double2 v = bs[j * 32];
      fb[buf][j][0] = v.x;
      fb[buf][j][1] = v.y;
      fb[buf][j][2] = v.x + v.y;  // Br + Bi
    }
  };

  int task = task0, slot = 0;
  unsigned ph = 0;
  long long tile = blockIdx.x;
  TmTile tt = tm_decode(descs, n_desc, task, tile);
  int ks_n = descs[task].Ko * ((descs[task].Ki + TM_BK - 1) / TM_BK);
  int ks = 0;
  mbar_wait(full0, 0);
  load_frag(0, 0, 0);
  for (;;) {
#pragma unroll
    for (int kq = 0; kq < TM_BK / 4; ++kq) {
      const int cur = kq & 1;
      if (kq + 1 < TM_BK / 4) {
        load_frag(cur ^ 1, slot, kq + 1);
      } else {
        // Every fragment of this slot has been read: hand the slot back.  The reads are generic-
        // proxy LDS and the next write to the slot is the producer's TMA (async proxy): without
        // a proxy fence the arrive could overtake LDS still queued (ptxas schedules the last
        // k-quad's LDS a few instructions before it), and a fast TMA overwrote the slot under
        // them about once per 20 C3 executes (one wrong fused-dot partial; tools/race_hunt.py).
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncwarp();
        if (lane == 0) mbar_arrive(empty0 + 8 * slot);
        if (++slot == TM_ST) { slot = 0; ph ^= 1; }
        if (ks + 1 < ks_n) {  // (the next tile's first fragments are loaded after the epilogue)
          mbar_wait(full0 + 8 * slot, ph);
          load_frag(cur ^ 1, slot, 0);
        }
      }
#pragma unroll
      for (int i = 0; i < MI; ++i)
#pragma unroll
        for (int j = 0; j < NJ; ++j) {
          dmma(acc[i][j][0][0], acc[i][j][0][1], fa[cur][i][0], fb[cur][j][0]);  // Ar·Br
          dmma(acc[i][j][1][0], acc[i][j][1][1], fa[cur][i][1], fb[cur][j][1]);  // Ai·Bi
          dmma(acc[i][j][2][0], acc[i][j][2][1], fa[cur][i][2], fb[cur][j][2]);  // (Ar+Ai)·(Br+Bi)
        }
    }
    const GemmDesc &dd = descs[task];
    if (dd.D && ks + 2 == ks_n) {
      // fused dot: pull this tile's partner block into L2 one stage before the epilogue
      const double2 *D = dd.D + tt.t * dd.sDt + tt.mo * dd.sDmo + tt.no * dd.sDno;
      const bool mrow = dd.sDni == 1;
      const int rows = mrow ? min(TM_BM, dd.Mi - tt.m0) : min(TM_BN, dd.Ni - tt.n0);
      const int segs = (mrow ? TM_BN : TM_BM) / 8;
      for (int q = tid; q < rows * segs; q += TM_NW * 32) {
        const int r = q / segs, seg = (q % segs) * 8;
        const double2 *pp = mrow ? D + (long long)(tt.m0 + r) * dd.sDmi + tt.n0 + seg
                                 : D + (long long)(tt.n0 + r) * dd.sDni + tt.m0 + seg;
        asm volatile("prefetch.global.L2 [%0];\n" ::"l"(pp));
      }
    }
    if (++ks < ks_n) continue;
    // ---- tile done: 3M combine, then store C or the fused dot's partial sum
    {
      const int Mi = dd.Mi, Ni = dd.Ni;
      auto cval = [&](int i, int j, int h, double &re, double &im) {
        re = acc[i][j][0][h] - acc[i][j][1][h];
        im = acc[i][j][2][h] - (acc[i][j][0][h] + acc[i][j][1][h]);
      };
      if (dd.D) {
        const double2 *D = dd.D + tt.t * dd.sDt + tt.mo * dd.sDmo + tt.no * dd.sDno;
        const long long sDmi = dd.sDmi, sDni = dd.sDni;
        double pr = 0.0, pim = 0.0;
        constexpr int CH = MI;  // partner rows in flight
#pragma unroll
        for (int i0 = 0; i0 < MI; i0 += CH) {
          double2 y[CH][NJ][2];
#pragma unroll
          for (int ii = 0; ii < CH; ++ii) {
            const int m = tt.m0 + wm * 32 + (i0 + ii) * 8 + (lane >> 2);
#pragma unroll
            for (int j = 0; j < NJ; ++j)
#pragma unroll
              for (int h = 0; h < 2; ++h) {
                const int n = tt.n0 + wn * 16 + j * 8 + (lane & 3) * 2 + h;
                y[ii][j][h] = (m < Mi && n < Ni) ? D[(long long)m * sDmi + (long long)n * sDni] : make_double2(0.0, 0.0);
              }
          }
#pragma unroll
          for (int ii = 0; ii < CH; ++ii)
#pragma unroll
            for (int j = 0; j < NJ; ++j)
#pragma unroll
              for (int h = 0; h < 2; ++h) {
                double re, im;
                cval(i0 + ii, j, h, re, im);
                pr += re * y[ii][j][h].x - im * y[ii][j][h].y;
                pim += re * y[ii][j][h].y + im * y[ii][j][h].x;
              }
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) {
          pr += __shfl_xor_sync(0xffffffffu, pr, off);
          pim += __shfl_xor_sync(0xffffffffu, pim, off);
        }
        if (lane == 0) dd.part[(tile - dd.tile_begin) * TM_NW + warp] = make_double2(pr, pim);
      } else {
        double2 *C = dd.C + tt.t * dd.sCt + tt.mo * dd.sCmo + tt.no * dd.sCno;
        const long long sCmi = dd.sCmi, sCni = dd.sCni;
#pragma unroll
        for (int i = 0; i < MI; ++i) {
          const int m = tt.m0 + wm * 32 + i * 8 + (lane >> 2);
          if (m >= Mi) continue;
#pragma unroll
          for (int j = 0; j < NJ; ++j) {
            const int n = tt.n0 + wn * 16 + j * 8 + (lane & 3) * 2;
            double2 *cp = C + (long long)m * sCmi + (long long)n * sCni;
            double re, im;
            cval(i, j, 0, re, im);
            if (n < Ni) cp[0] = make_double2(re, im);
            cval(i, j, 1, re, im);
            if (n + 1 < Ni) cp[sCni] = make_double2(re, im);
          }
        }
      }
    }
#pragma unroll
    for (int i = 0; i < MI; ++i)
#pragma unroll
      for (int j = 0; j < NJ; ++j)
#pragma unroll
        for (int q = 0; q < 3; ++q) acc[i][j][q][0] = acc[i][j][q][1] = 0.0;
    if ((tile += G) >= total) break;
    tt = tm_decode(descs, n_desc, task, tile);
    ks_n = descs[task].Ko * ((descs[task].Ki + TM_BK - 1) / TM_BK);
    ks = 0;
    mbar_wait(full0 + 8 * slot, ph);
    load_frag(0, slot, 0);
  }
}

// ---------------------------------------------------------------- dot / trace

constexpr int DT = 256;

__device__ __forceinline__ void cmac(double &sr, double &si, double2 a, double2 b) {
  sr += a.x * b.x - a.y * b.y;
  si += a.x * b.y + a.y * b.x;
}

constexpr int DOT_MINB = 3;    // resident dot CTAs per SM the register budget is sized for
constexpr int DOT_UNROLL = 2;  // mode-1 micro-block pairs in flight per thread

// one complex element, read once: no L1 allocation (C4 dots 55.7 → 48.4 ms, round 1)
__device__ __forceinline__ double2 ldg_stream(const double2 *p) {
  double2 v;
  asm("ld.global.nc.L1::no_allocate.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  return v;
}

// 32 bytes (two complex elements) in one LDG.E.256 (sm_100); p must be 32-byte aligned
__device__ __forceinline__ void ldg_pair(const double2 *p, double2 &a, double2 &b) {
  asm("ld.global.nc.L1::no_allocate.v4.f64 {%0, %1, %2, %3}, [%4];"
      : "=d"(a.x), "=d"(a.y), "=d"(b.x), "=d"(b.y)
      : "l"(p));
}

// mode 1: s = Σ_o Σ_{y<Y} Σ_{x<X} A[o][y·sAy + x] · B[o][x·sBx + y]   (layout.cpp: sAx = sBy = 1)
// Register-only transpose: a thread owns a 2×2 (y, x) micro-block and loads A[y..y+1][x..x+1]
// and B[x..x+1][y..y+1], so every pair A[y][x]·B[x][y] meets in one thread: no shared-memory
// staging, no barrier.  A warp covers 16 y × 8 x, so each load instruction reads 8 whole
// 128-byte lines.  V256 (every row start and x even, pointers 32-byte aligned): a thread's
// two elements of a row come in one 32-byte LDG.E.256 — half the load instructions and L1
// wavefronts of two 16-byte loads, whose half-sector pattern kept l1tex 92% busy on C4.
// DOT_UNROLL blocks keep 4·DOT_UNROLL (V256) or 8·DOT_UNROLL loads in flight per thread.
// Slices are < 2^31 elements (executor.cu guard): 32-bit offsets.
template <bool V256>
__device__ __forceinline__ void zdot_mode1(const DotDesc &d, const double2 *__restrict__ A,
                                           const double2 *__restrict__ B, int tid, double &sr, double &si) {
  const int lane = tid & 31, w = tid >> 5;
  const int ty = lane >> 2, tx = lane & 3;
  const int X = d.X, Y = d.Y;
  const int nxb = (X + 7) >> 3, per_o = ((Y + 15) >> 4) * nxb;
  const int O1 = d.O[1], O2 = d.O[2];
  const int nb = d.O[0] * O1 * O2 * per_o;
  const int sAy = (int)d.sAy, sBx = (int)d.sBx;
  constexpr int NW = DT / 32;
  for (int b0 = w; b0 < nb; b0 += NW * DOT_UNROLL) {
    double2 va[DOT_UNROLL][4], vb[DOT_UNROLL][4];
#pragma unroll
    for (int u = 0; u < DOT_UNROLL; ++u) {
      const int b = b0 + u * NW;
      const int o = b / per_o, r = b - o * per_o;
      const int yb = r / nxb, xb = r - yb * nxb;
      const int o2 = o % O2, o01 = o / O2, o1 = o01 % O1, o0 = o01 / O1;
      const int offA = (int)(o0 * d.sAo[0] + o1 * d.sAo[1] + o2 * d.sAo[2]);
      const int offB = (int)(o0 * d.sBo[0] + o1 * d.sBo[1] + o2 * d.sBo[2]);
      const int y = yb * 16 + 2 * ty, x = xb * 8 + 2 * tx;
      const bool in = b < nb;
      if constexpr (V256) {  // X, Y even: the pair (x, x + 1) is in or out together
        const bool v = in && y < Y && x < X;
        const double2 z = make_double2(0.0, 0.0);
        va[u][0] = va[u][1] = va[u][2] = va[u][3] = z;
        vb[u][0] = vb[u][1] = vb[u][2] = vb[u][3] = z;
        if (v) {
          ldg_pair(A + offA + y * sAy + x, va[u][0], va[u][1]);        // A[y][x], A[y][x+1]
          ldg_pair(A + offA + (y + 1) * sAy + x, va[u][2], va[u][3]);  // A[y+1][x], A[y+1][x+1]
          ldg_pair(B + offB + x * sBx + y, vb[u][0], vb[u][2]);        // B[x][y], B[x][y+1]
          ldg_pair(B + offB + (x + 1) * sBx + y, vb[u][1], vb[u][3]);  // B[x+1][y], B[x+1][y+1]
        }
      } else {
#pragma unroll
        for (int i = 0; i < 2; ++i)
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            const bool v = in && y + i < Y && x + j < X;
            // (16-byte halves of one sector: the second is an L1 hit, so L1 allocation stays)
            va[u][2 * i + j] = v ? __ldg(A + offA + (y + i) * sAy + x + j) : make_double2(0.0, 0.0);
            vb[u][2 * i + j] = v ? __ldg(B + offB + (x + j) * sBx + y + i) : make_double2(0.0, 0.0);
          }
      }
    }
#pragma unroll
    for (int u = 0; u < DOT_UNROLL; ++u)
#pragma unroll
      for (int k = 0; k < 4; ++k) cmac(sr, si, va[u][k], vb[u][k]);
  }
}

__device__ __forceinline__ void zdot_body(const DotDesc *__restrict__ descs, int n_desc) {
  __shared__ double red[2][DT / 32];
  // Slice-major CTA order (every task of the launch has Lt CTAs): the CTAs resident at any
  // moment cover a few slices of every dot, so an operand shared by several dots of the launch
  // (C4's c = 2 products are each read by ~70 dots) is read from DRAM once per slice and
  // served from L2 afterwards; task-major order kept whole operands live and re-read them.
  const long long cta = blockIdx.x;
  const int t = (int)(cta / n_desc);
  const DotDesc &d = descs[cta - (long long)t * n_desc];
  const int tid = threadIdx.x;
  const double2 *A = d.A + t * d.sAt;
  const double2 *B = d.B ? d.B + t * d.sBt : nullptr;
  double sr = 0.0, si = 0.0;
  if (d.mode == 0) {  // x runs contiguous in both operands: rows o, threads along x
    const int X = d.X, O1 = d.O[1], O2 = d.O[2], Ot = d.O[0] * O1 * O2;
    const int sAx = (int)d.sAx, sBx = (int)d.sBx;
    if (X >= DT / 2) {
      for (int o = 0; o < Ot; ++o) {
        const int o2 = o % O2, o01 = o / O2, o1 = o01 % O1, o0 = o01 / O1;
        const double2 *Ao = A + (o0 * d.sAo[0] + o1 * d.sAo[1] + o2 * d.sAo[2]);
        const double2 *Bo = B + (o0 * d.sBo[0] + o1 * d.sBo[1] + o2 * d.sBo[2]);
#pragma unroll 8
        for (int x = tid; x < X; x += DT) cmac(sr, si, ldg_stream(Ao + x * sAx), ldg_stream(Bo + x * sBx));
      }
    } else {  // short runs: flat (o, x) index, 32-bit decode per element
      const int total = Ot * X;
#pragma unroll 4
      for (int e = tid; e < total; e += DT) {
        const int o = e / X, x = e - o * X;
        const int o2 = o % O2, o01 = o / O2, o1 = o01 % O1, o0 = o01 / O1;
        const int offA = (int)(o0 * d.sAo[0] + o1 * d.sAo[1] + o2 * d.sAo[2]) + x * sAx;
        const int offB = (int)(o0 * d.sBo[0] + o1 * d.sBo[1] + o2 * d.sBo[2]) + x * sBx;
        cmac(sr, si, ldg_stream(A + offA), ldg_stream(B + offB));
      }
    }
  } else {
    // 32-byte pair loads need even row starts and x; the descriptor fixes this per dot
    const bool v256 = ((((unsigned long long)A | (unsigned long long)B) & 31ull) == 0) &&
                      (((d.X | d.Y | d.sAy | d.sBx | d.sAo[0] | d.sAo[1] | d.sAo[2] | d.sBo[0] | d.sBo[1] |
                         d.sBo[2]) & 1) == 0);
    if (v256) zdot_mode1<true>(d, A, B, tid, sr, si);
    else zdot_mode1<false>(d, A, B, tid, sr, si);
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

// Dots of one launch that share their A operand (C4: each c = 2 product is the A side of many
// final dots), for slices of ≤ kDotGroupElems complex with no outer index: one CTA per (group of
// ≤ kDotGroupPartners such dots, slice) stages A's slice in shared memory once, in the order its
// partners are read, and streams the partners B against it, one element of every partner in
// flight together.  The C4 dot launches were L2-bound (11.6 TB/s served by L2 for 512 MB from
// DRAM, profiles/r02/ncu_dot_c4_r02.json); staging the shared side cuts their L2 bytes.  Groups
// are formed inside plan-order batches (a launch covers the same operands as an ungrouped one).
// Measured on C4 (profiles/r02/dotgroup/): 6 partners at 2 CTAs/SM 49.2 → 43.3 ms of dots per
// step; 8 partners (larger groups, fewer CTAs) and 2-4 partners at 3 CTAs/SM were slower.
// Element order, per-thread sums and the reduction tree depend only on the descriptor, never
// on the group it lands in, so a dot's value is bitwise the same whatever the grouping (GPU
// counts, windows and batch boundaries change the groups).
//   term (x, y) = A[y·sAy + x·sAx] · B[x·sBx + y·sBy],  e = x·Y + y enumerates B (sBy = 1 in
//   mode 1; Y = 1 in mode 0, where x runs contiguous in both)
// smem S[x·P + y] = A[y][x], P = Y + 1 when Y > 1 (conflict-free transposed staging stores).
__global__ void __launch_bounds__(DT, 2) zdot_group_kernel(const __grid_constant__ DotGroupBatch b) {
  extern __shared__ __align__(16) double2 S[];
  __shared__ double2 red[kDotGroupPartners][DT / 32];
  const int ng = b.n_groups;
  const int t = (int)(blockIdx.x / ng), g = (int)(blockIdx.x - (unsigned)t * ng);  // slice-major
  const int i0 = b.first[g], np = b.first[g + 1] - i0;
  const DotDesc &d0 = b.d[i0];
  const int X = d0.X, Y = d0.Y, P = Y > 1 ? Y + 1 : 1, XY = X * Y;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  {
    const double2 *A = d0.A + t * d0.sAt;
    const int sAy = (int)d0.sAy, sAx = (int)d0.sAx;
#pragma unroll 8
    for (int e = tid; e < XY; e += DT) {  // coalesced along x (sAx = 1)
      const int y = e / X, x = e - y * X;
      S[x * P + y] = ldg_stream(A + y * sAy + x * sAx);
    }
  }
  const double2 *Bp[kDotGroupPartners];  // (a group shares the partners' strides too)
#pragma unroll
  for (int p = 0; p < kDotGroupPartners; ++p) Bp[p] = b.d[i0 + (p < np ? p : 0)].B + t * d0.sBt;
  const int sBx = (int)d0.sBx, sBy = (int)d0.sBy;
  double sr[kDotGroupPartners], si[kDotGroupPartners];
#pragma unroll
  for (int p = 0; p < kDotGroupPartners; ++p) sr[p] = si[p] = 0.0;
  __syncthreads();
#pragma unroll 2
  for (int e = tid; e < XY; e += DT) {  // every partner's element e in flight together
    const int x = e / Y, y = e - x * Y;
    const double2 a = S[x * P + y];
#pragma unroll
    for (int p = 0; p < kDotGroupPartners; ++p)
      if (p < np) cmac(sr[p], si[p], a, ldg_stream(Bp[p] + x * sBx + y * sBy));
  }
#pragma unroll
  for (int p = 0; p < kDotGroupPartners; ++p) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      sr[p] += __shfl_xor_sync(0xffffffffu, sr[p], off);
      si[p] += __shfl_xor_sync(0xffffffffu, si[p], off);
    }
    if (lane == 0) red[p][warp] = make_double2(sr[p], si[p]);
  }
  __syncthreads();
  if (tid < np) {  // warps in order (the same tree as zdot_body)
    double ar = 0.0, ai = 0.0;
    for (int w = 0; w < DT / 32; ++w) { ar += red[tid][w].x; ai += red[tid][w].y; }
    b.d[i0 + tid].out[t] = make_double2(ar, ai);
  }
}

// One warp per (dot, slice) for the short reductions (2: meson trace, 3: sum of the fused
// GEMM's partials): no block barrier, a fixed-order butterfly (deterministic).  The flat
// dots (mode 0) stay on the CTA kernel: a warp per C4 64×64 dot put 8× more slices in
// flight, the working set outgrew L2 and the dots took 177 instead of 83 ms per step.
constexpr int DW = DT / 32;  // items per CTA

__device__ __forceinline__ void zdot_warp_body(const DotDesc *__restrict__ descs, int n_desc, long long items) {
  const long long item = (long long)blockIdx.x * DW + (threadIdx.x >> 5);
  if (item >= items) return;
  const int t = (int)(item / n_desc);
  const DotDesc &d = descs[item - (long long)t * n_desc];
  const int lane = threadIdx.x & 31;
  const double2 *A = d.A + t * d.sAt;
  double sr = 0.0, si = 0.0;
  if (d.mode == 3) {
    for (int i = lane; i < d.X; i += 32) {
      const double2 a = A[i];
      sr += a.x;
      si += a.y;
    }
  } else {  // mode 2
    for (int i = lane; i < d.X; i += 32) {
      const double2 a = A[(long long)i * d.sAx];
      sr += a.x;
      si += a.y;
    }
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    sr += __shfl_xor_sync(0xffffffffu, sr, off);
    si += __shfl_xor_sync(0xffffffffu, si, off);
  }
  if (lane == 0) d.out[t] = make_double2(sr, si);
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
template <bool AKF, bool BNF>
__global__ void __launch_bounds__(128, 2) zgemm_persistent(const __grid_constant__ GemmBatch b, long long total) {
  zgemm_persistent_body<2, 2, 32, 16, AKF, BNF>(b.d, b.n, total);
}

__global__ void __launch_bounds__(128, 2) zgemm_persistent_kb(const __grid_constant__ GemmBatch b, long long total) {
  zgemm_persistent_body<2, 2, 32, 16, true, true, true>(b.d, b.n, total);
}

// The persistent GEMM for layout class cls (0..3 = (A contiguous along m ? 2 : 0) +
// (B contiguous along k ? 1 : 0), layout.cpp gemm_class).
void (*persistent_fn(int cls))(const GemmBatch, long long) {
  switch (cls) {
    case 0: return zgemm_persistent<true, true>;
    case 1: return zgemm_persistent<true, false>;
    case 2: return zgemm_persistent<false, true>;
    default: return zgemm_persistent<false, false>;
  }
}

template <bool AK, bool BK>
__global__ void __launch_bounds__(TM_THREADS, 1) zgemm_tma(const __grid_constant__ GemmTmaBatch b, long long total) {
  zgemm_tma_body<AK, BK>(b, total);
}

__global__ void __launch_bounds__(DT, DOT_MINB) zdot_kernel(const __grid_constant__ DotBatch b) { zdot_body(b.d, b.n); }
__global__ void __launch_bounds__(DT) zdot_warp_kernel(const __grid_constant__ DotBatch b, long long items) {
  zdot_warp_body(b.d, b.n, items);
}

// FP64 tensor-pipe ceiling probe: register-only DMMA chains (8 independent accumulators per
// warp hide the DMMA latency), no memory traffic.  512 flops per DMMA.8x8x4.
__global__ void __launch_bounds__(128) dmma_probe_kernel(double *out, int iters) {
  double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4;
  double c[8][2];
#pragma unroll
  for (int i = 0; i < 8; ++i) c[i][0] = c[i][1] = 0.0;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) dmma(c[i][0], c[i][1], a, b);
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) s += c[i][0] + c[i][1];
  if (s == 12345.678) out[0] = s;  // (never true: keeps the chains live)
}

}  // namespace

cudaError_t probe_fp64_peak(double seconds, double *burst_tflops, double *sustained_tflops) {
  int dev = 0, sms = 148;
  cudaError_t e;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  double *out = nullptr;
  if ((e = cudaMalloc(&out, 8)) != cudaSuccess) return e;
  cudaStream_t st;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int iters = 4096, ctas = sms * 4;  // 4 CTAs × 4 warps = 16 warps per SM
  const double flops = 512.0 * 8 * iters * (double)ctas * 4;
  float best = 1e30f;
  for (int rep = 0; rep < 5; ++rep) {  // burst: the best of a few single launches
    cudaEventRecord(e0, st);
    dmma_probe_kernel<<<ctas, 128, 0, st>>>(out, iters);
    cudaEventRecord(e1, st);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms > 0 && ms < best) best = ms;
  }
  *burst_tflops = flops / (best * 1e-3) * 1e-12;
  const int n = std::max(1, (int)(seconds / (best * 1e-3)));
  cudaEventRecord(e0, st);
  for (int i = 0; i < n; ++i) dmma_probe_kernel<<<ctas, 128, 0, st>>>(out, iters);
  cudaEventRecord(e1, st);
  cudaEventSynchronize(e1);
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  *sustained_tflops = flops * n / (ms * 1e-3) * 1e-12;
  e = cudaGetLastError();
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaStreamDestroy(st);
  cudaFree(out);
  return e;
}

void gemm_tile_shape(int cls, int *bm, int *bn) {
  *bm = 64;
  *bn = 32;
  if (cls >= kGemmClassTMA) { *bm = TM_BM; *bn = TM_BN; return; }
  if (cls == 4) *bn = 64;  // per-tile gather kernel
}

bool gemm_uses_3m(int cls) { return cls != 4; }

int gemm_warps_per_tile(int cls) { return cls >= kGemmClassTMA ? TM_NW : 4; }

int gemm_kernel_class(int layout_cls, int Ko) {
  // class 4 (no unit stride on an operand's free or inner contracted index) goes to the
  // blocked-K persistent kernel when the outer contracted index is long enough to fill a
  // 4 × 4 k-block; else to the per-tile gather kernel
  if (layout_cls == 4 && Ko >= 4) return kGemmClassKB;
  return layout_cls;
}

cudaError_t launch_gemm_group(const GemmBatch *b, long long total_tiles, int cls, cudaStream_t st) {
  // (one host thread launches: the executor replays the plan sequentially)
  // The shared-memory opt-in is recorded per device context: track it per device, so the
  // persistent GEMMs on a second (third, ...) device of one process get it too.
  static unsigned long long attr_set = 0;  // bit d: set on device d
  int cur_dev = 0;
  if (cudaError_t e = cudaGetDevice(&cur_dev); e != cudaSuccess) return e;
  const unsigned long long dev_bit = 1ull << (cur_dev & 63);
  if (!(attr_set & dev_bit)) {
    cudaError_t e = cudaFuncSetAttribute(zgemm_dmma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, GEMM_SMEM);
    if (e != cudaSuccess) return e;
    for (int c = 0; c < 4; ++c) {
      e = cudaFuncSetAttribute(persistent_fn(c), cudaFuncAttributeMaxDynamicSharedMemorySize, PCfg<64, 32>::SMEM);
      if (e != cudaSuccess) return e;
    }
    e = cudaFuncSetAttribute(zgemm_persistent_kb, cudaFuncAttributeMaxDynamicSharedMemorySize, PCfg<64, 32>::SMEM);
    if (e != cudaSuccess) return e;
    attr_set |= dev_bit;
  }
  if (total_tiles <= 0) return cudaSuccess;
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, cur_dev);
  if (cls == 4) {  // per-tile kernel; gathers operands with no unit-stride free or inner contracted index
    long long grid = total_tiles < (1LL << 30) ? total_tiles : (1LL << 30);
    zgemm_dmma_kernel<<<(unsigned)grid, NT, GEMM_SMEM, st>>>(*b, total_tiles);
    return cudaGetLastError();
  }
  long long grid = 2LL * sms;  // 2 resident CTAs per SM
  if (grid > total_tiles) grid = total_tiles;
  if (cls == kGemmClassKB)  // blocked-K gather (gemm_kernel_class)
    zgemm_persistent_kb<<<(unsigned)grid, 128, PCfg<64, 32>::SMEM, st>>>(*b, total_tiles);
  else
    persistent_fn(cls)<<<(unsigned)grid, 128, PCfg<64, 32>::SMEM, st>>>(*b, total_tiles);
  return cudaGetLastError();
}

bool gemm_tma_class(const GemmDesc &d, int *cls) {
  const bool ak = d.sAki == 1, bk = d.sBki == 1;  // K-major operands (else contiguous along m / n)
  if (!ak && d.sAmi != 1) return false;
  if (!bk && d.sBni != 1) return false;
  if (d.Ki % 4 != 0) return false;  // k-quads are the maps' inner unit
  // 5 dimensions per map: K-major (k4, row, kq, t, outer-or-ko), MN-major (row pair, k4, row/2, kq, t)
  if (ak ? (d.Ko > 1 && d.Mo > 1) : (d.Ko > 1 || d.Mo > 1 || d.Mi % 2 != 0)) return false;
  if (bk ? (d.Ko > 1 && d.No > 1) : (d.Ko > 1 || d.No > 1 || d.Ni % 2 != 0)) return false;
  if ((((uintptr_t)d.A) | ((uintptr_t)d.B)) & 15) return false;
  // The TMA kernel's tile is 128 rows: a short M (C4/C5's single N = 64 leg, C1's N = 32)
  // would leave most of it zero-filled; the 64-row cp.async kernel takes those (C5 at its
  // stated size: 8.4 s per step on the 128-row tile against 6.9 s).
  const int tm = (d.Mi + TM_BM - 1) / TM_BM * TM_BM;
  if (8 * tm > 9 * d.Mi) return false;  // more than 1/9 of the tile's rows wasted
  *cls = kGemmClassTMA + (ak ? 0 : 2) + (bk ? 1 : 0);
  return true;
}

namespace {
PFN_cuTensorMapEncodeTiled_v12000 tensor_map_encoder() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = [] {
    void *f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      f = nullptr;
    return (PFN_cuTensorMapEncodeTiled_v12000)f;
  }();
  return fn;
}

// One operand's map.  rows/srow: its free index inside the tile (m or n) and stride; sk: the
// inner contracted stride; Ki; Lt and the slice stride; outer: (size, stride) of the 5th
// K-major dimension (Ko when > 1, else the operand's outer free index).  Strides in complex.
bool encode_operand(CUtensorMap *m, const double2 *base, bool kmaj, int rows, long long srow, long long sk, int Ki,
                    int Lt, long long st, int box_rows, long long outer_n, long long outer_s) {
  auto enc = tensor_map_encoder();
  if (!enc) return false;
  cuuint64_t dims[5], str[4];
  cuuint32_t box[5], es[5] = {1, 1, 1, 1, 1};
  if (kmaj) {  // (k4 as 8 doubles, row, kq, t, outer) → smem [kq][row][k4]
    dims[0] = 8; dims[1] = rows; dims[2] = Ki / 4; dims[3] = Lt; dims[4] = outer_n;
    str[0] = srow * 16; str[1] = 64; str[2] = st * 16; str[3] = (outer_n > 1 ? outer_s : 1) * 16;
    box[0] = 8; box[1] = box_rows; box[2] = TM_BK / 4; box[3] = 1; box[4] = 1;
  } else {     // (row pair as 4 doubles, k4, row/2, kq, t) → smem [kq][row/2][k4][2]
    dims[0] = 4; dims[1] = 4; dims[2] = rows / 2; dims[3] = Ki / 4; dims[4] = Lt;
    str[0] = sk * 16; str[1] = 32; str[2] = sk * 4 * 16; str[3] = st * 16;
    box[0] = 4; box[1] = 4; box[2] = box_rows / 2; box[3] = TM_BK / 4; box[4] = 1;
  }
  for (int i = 0; i < 4; ++i)
    if (str[i] == 0 || str[i] % 16 != 0 || str[i] >= (1ull << 40)) return false;
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 5, (void *)base, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
             CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
}  // namespace

bool gemm_tma_encode(const GemmDesc &d, int cls, CUtensorMap *a, CUtensorMap *b) {
  const int c = cls - kGemmClassTMA;
  const bool ak = (c & 2) == 0, bk = (c & 1) != 0;
  const long long aon = d.Ko > 1 ? d.Ko : d.Mo, aos = d.Ko > 1 ? d.sAko : d.sAmo;
  const long long bon = d.Ko > 1 ? d.Ko : d.No, bos = d.Ko > 1 ? d.sBko : d.sBno;
  return encode_operand(a, d.A, ak, d.Mi, ak ? d.sAmi : 1, ak ? 1 : d.sAki, d.Ki, d.Lt, d.sAt, TM_BM, aon, aos) &&
         encode_operand(b, d.B, bk, d.Ni, bk ? d.sBni : 1, bk ? 1 : d.sBki, d.Ki, d.Lt, d.sBt, TM_BN, bon, bos);
}

cudaError_t launch_gemm_tma_group(const GemmTmaBatch *b, long long total_tiles, int cls, cudaStream_t st) {
  static unsigned long long attr_set = 0;  // per device (see launch_gemm_group)
  int dev = 0;
  if (cudaError_t e = cudaGetDevice(&dev); e != cudaSuccess) return e;
  const unsigned long long bit = 1ull << (dev & 63);
  if (!(attr_set & bit)) {
    for (auto fn : {zgemm_tma<true, true>, zgemm_tma<true, false>, zgemm_tma<false, true>, zgemm_tma<false, false>}) {
      cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, TM_SMEM);
      if (e != cudaSuccess) return e;
    }
    attr_set |= bit;
  }
  if (total_tiles <= 0) return cudaSuccess;
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  long long grid = sms;  // one resident CTA per SM (TM_NW consumer warps + the producer)
  if (grid > total_tiles) grid = total_tiles;
  switch (cls - kGemmClassTMA) {
    case 0: zgemm_tma<true, false><<<(unsigned)grid, TM_THREADS, TM_SMEM, st>>>(*b, total_tiles); break;
    case 1: zgemm_tma<true, true><<<(unsigned)grid, TM_THREADS, TM_SMEM, st>>>(*b, total_tiles); break;
    case 2: zgemm_tma<false, false><<<(unsigned)grid, TM_THREADS, TM_SMEM, st>>>(*b, total_tiles); break;
    default: zgemm_tma<false, true><<<(unsigned)grid, TM_THREADS, TM_SMEM, st>>>(*b, total_tiles); break;
  }
  return cudaGetLastError();
}

cudaError_t launch_dot_group(const DotBatch *b, long long total_ctas, int cls, cudaStream_t st) {
  if (total_ctas <= 0) return cudaSuccess;
  if (cls == 0) {  // modes 2, 3: a warp per (dot, slice)
    zdot_warp_kernel<<<(unsigned)((total_ctas + DW - 1) / DW), DT, 0, st>>>(*b, total_ctas);
    return cudaGetLastError();
  }
  zdot_kernel<<<(unsigned)total_ctas, DT, 0, st>>>(*b);
  return cudaGetLastError();
}

bool dot_groupable(const DotDesc &d) {
  if (!(d.mode == 0 || d.mode == 1) || !d.B) return false;
  if (d.O[0] * d.O[1] * d.O[2] != 1 || d.sAx != 1) return false;
  if ((long long)d.X * d.Y > kDotGroupElems) return false;
  return d.mode == 0 ? (d.Y == 1 && d.sBx == 1) : d.sBy == 1;
}

static size_t dot_group_smem(int X, int Y) { return (size_t)X * (Y > 1 ? Y + 1 : 1) * sizeof(double2); }

cudaError_t launch_dot_shared_group(const DotGroupBatch *b, int Lt, cudaStream_t st) {
  static unsigned long long attr_set = 0;  // per device (see launch_gemm_group)
  int dev = 0;
  if (cudaError_t e = cudaGetDevice(&dev); e != cudaSuccess) return e;
  const unsigned long long bit = 1ull << (dev & 63);
  if (!(attr_set & bit)) {
    cudaError_t e = cudaFuncSetAttribute(zdot_group_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)dot_group_smem(64, 64));
    if (e != cudaSuccess) return e;
    attr_set |= bit;
  }
  if (b->n_groups <= 0 || Lt <= 0) return cudaSuccess;
  size_t smem = 0;  // the largest group of the batch
  for (int g = 0; g < b->n_groups; ++g) {
    const DotDesc &d = b->d[b->first[g]];
    smem = std::max(smem, dot_group_smem(d.X, d.Y));
  }
  zdot_group_kernel<<<(unsigned)((long long)b->n_groups * Lt), DT, smem, st>>>(*b);
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
