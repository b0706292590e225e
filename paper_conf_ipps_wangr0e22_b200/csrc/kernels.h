// kernels.h — device-side task descriptors and launchers of the contraction kernels
// (sm_100a).  Complex doubles are stored interleaved (double2 = re, im) everywhere on the
// device, the layout of the C-ABI, so no conversion pass exists.
#pragma once

#include <cstdint>
#include <cuda.h>  // CUtensorMap (the type only: tensor maps are encoded through the runtime's driver entry point)
#include <cuda_runtime.h>

namespace micco {

// A pairwise hadron contraction with a rank >= 1 result, as a batched GEMM over the time
// slices ("batched matrix multiplications for a meson system or batched
// tensor contractions for a baryon system"):
//   C[t][mo,mi][no,ni] = Σ_{ko,ki} A[t][mo,mi][ko,ki] · B[t][ko,ki][no,ni]
// Every index is split into an outer part (grid / loop) and an inner part (tiled), each
// with its own stride per tensor, so permuted operand legs (op(A) ∈ {N, T}, baryon legs in
// any position) are read in place without transposes.  Strides are in complex elements.
struct GemmDesc {
  const double2 *A;
  const double2 *B;
  double2 *C;
  long long sAt, sBt, sCt;
  int Mo, Mi, No, Ni, Ko, Ki;
  long long sAmo, sAmi, sAko, sAki;
  long long sBko, sBki, sBno, sBni;
  long long sCmo, sCmi, sCno, sCni;
  int Lt, tilesM, tilesN, cls;  // cls: operand layout class (gemm_layout_class)
  long long tile_begin;  // first CTA tile of this task in the grouped launch
  // Fused final contraction (GEMM → dot, SURVEY.md §8(a) A9 "fused into the last GEMM's
  // epilogue"): when D != nullptr, C is never written; instead every consumer warp writes
  //   part[(task tile) * 4 + warp] = Σ_{its (m, n)} C[t][m][n] · D[t][m·sD_m + n·sD_n]
  // and a fixed-order partial sum (zdot mode 3) produces the scalar per slice.
  const double2 *D;
  double2 *part;
  long long sDt, sDmo, sDmi, sDno, sDni;
};

// The final reduction of two nodes to a scalar per slice ("until
// only two hadrons are left"), s_t = Σ_idx A[t][idx] · B[t][π(idx)], or a meson trace
// s_t = Σ_i A[t][i][i] when B == nullptr.
//   mode 0: x is contiguous in both A and B (flat run of X elements per outer index)
//   mode 1: x contiguous in A, y contiguous in B → 32×32 shared-memory transpose tiles
//   mode 2: trace (stride sAx along x)
//   mode 3: Σ_x A[x] (fixed-order sum of X partials of a fused GEMM → dot)
struct DotDesc {
  const double2 *A;
  const double2 *B;
  double2 *out;          // out[t], t = 0..Lt-1 (a row of the scalar table)
  long long sAt, sBt;
  int mode, nO, X, Y;
  long long sAx, sAy, sBx, sBy;
  int O[3], pad0;
  long long sAo[3], sBo[3];
  int Lt, pad1;
  long long cta_begin;   // (unused by the kernel: CTA = t * n_desc + task, one per slice)
};

constexpr int kGemmBM = 64, kGemmBN = 64, kGemmBK = 8, kGemmStages = 4, kGemmThreads = 128;

// A grouped launch's descriptors, passed by value as one __grid_constant__ kernel parameter
// (≤ 32 KB of parameters per launch on sm_100).
constexpr int kGemmBatch = 128, kDotBatch = 192;
struct GemmBatch {
  int n, pad;
  GemmDesc d[kGemmBatch];
};
struct DotBatch {
  int n, pad;
  DotDesc d[kDotBatch];
};
static_assert(sizeof(GemmBatch) <= 32764 && sizeof(DotBatch) <= 32764, "kernel parameter limit");

// GEMM descriptors carry their operand-layout class (layout.h gemm_class): 0..3 = unit-stride
// inner index for both operands (warp-specialized kernel), 4 = generic gather kernel.
// 5 = class 4 on the blocked-K persistent kernel (gemm_kernel_class).
constexpr int kGemmClassKB = 5;
// 6..9 = the TMA warp-specialized kernel, kGemmClassTMA + (A contiguous along m ? 2 : 0) +
// (B contiguous along k ? 1 : 0), for contractions whose operands fit its tensor maps
// (gemm_tma_class); everything else stays on classes 0..5.
constexpr int kGemmClassTMA = 6, kGemmClasses = 10;

// A grouped launch of the TMA kernel: two tensor maps per descriptor (A, B), 64-byte aligned
// inside the __grid_constant__ parameter, then the descriptors.
constexpr int kGemmTmaBatch = 48;
struct GemmTmaBatch {
  CUtensorMap map[2 * kGemmTmaBatch];
  int n, pad[15];
  GemmDesc d[kGemmTmaBatch];
};
static_assert(sizeof(GemmTmaBatch) <= 32764, "kernel parameter limit");

// The TMA class of a descriptor (its strides and extents set, tile counts not yet), or false
// when its operands do not fit the kernel's 5-D tensor maps (then it keeps its class).
bool gemm_tma_class(const GemmDesc &d, int *cls);
// Encode the two operand tensor maps of a TMA-class descriptor (host; no device work).
bool gemm_tma_encode(const GemmDesc &d, int cls, CUtensorMap *a, CUtensorMap *b);

// The CTA tile (complex elements) of a kernel class; tilesM/tilesN of a descriptor must use it.
void gemm_tile_shape(int cls, int *bm, int *bn);
bool gemm_uses_3m(int cls);  // 3 DMMA products per complex MAC for this layout class
int gemm_warps_per_tile(int cls);  // fused-dot partial sums per tile (one per consumer warp)
int gemm_kernel_class(int layout_cls, int Ko);  // the launch class of a descriptor

// Grouped launches: descs in device memory (all of one layout class); grid covers the tiles.
cudaError_t launch_gemm_group(const GemmBatch *b, long long total_tiles, int cls, cudaStream_t st);
cudaError_t launch_gemm_tma_group(const GemmTmaBatch *b, long long total_tiles, int cls, cudaStream_t st);
// cls 0: a warp per dot and slice (modes 2, 3); cls 1: a CTA per dot and slice (modes 0, 1).
// total_ctas = Σ Lt over the batch (one work item per dot and slice).
inline int dot_class(int mode) { return mode == 0 || mode == 1 ? 1 : 0; }
cudaError_t launch_dot_group(const DotBatch *b, long long total_ctas, int cls, cudaStream_t st);

// Dots that share their A operand, launched as groups (kernels.cu zdot_group_kernel): the
// descriptors of a group are consecutive and share A (pointer, strides, extents) and the
// partners' strides; first[g] is the first descriptor of group g, first[n_groups] = n; a group
// holds at most kDotGroupPartners descriptors.  Only small slices without outer indices qualify
// (dot_groupable); the rest stay on launch_dot_group.
constexpr int kDotGroupBatch = 184, kDotGroupElems = 4096, kDotGroupPartners = 6;
struct DotGroupBatch {
  int n, n_groups;
  short first[kDotGroupBatch + 2];
  DotDesc d[kDotGroupBatch];
};
static_assert(sizeof(DotGroupBatch) <= 32764, "kernel parameter limit");
bool dot_groupable(const DotDesc &d);
cudaError_t launch_dot_shared_group(const DotGroupBatch *b, int Lt, cudaStream_t st);

// vals[g][t] = Π_{c in comps(g)} S[slot_c][t] (component scalars)
cudaError_t launch_finalize(int G, int Lt, const int *comp_off, const int *comp_slot,
                            const double2 *scalars, double2 *vals, cudaStream_t st);
// corr[t] = Σ_g coef_g · vals[g][t], fixed-order (deterministic for any GPU count)
cudaError_t launch_correlator_sum(int G, int Lt, const double2 *coefs, const double2 *vals,
                                  double2 *corr, cudaStream_t st);
// dst[i] += src[i] (exact: each slot is nonzero on exactly one source)
cudaError_t launch_accumulate(double2 *dst, const double2 *src, long long n, cudaStream_t st);

// FP64 DMMA ceiling of the current device (micco_probe_fp64_peak)
cudaError_t probe_fp64_peak(double seconds, double *burst_tflops, double *sustained_tflops);

}  // namespace micco
