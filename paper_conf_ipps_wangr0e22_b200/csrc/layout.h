// layout.h — index maps from a pairwise contraction (operand ranks, dims, contracted leg
// pairs) to the strided batched-GEMM / dot descriptors of kernels.h.  Pure host code, used
// by the builder (to reject layouts the kernels cannot read in place) and by the executor.
#pragma once

#include <cstdint>

namespace micco {

struct GemmLayout {
  int Mo, Mi, No, Ni, Ko, Ki;
  long long sAmo, sAmi, sAko, sAki;
  long long sBko, sBki, sBno, sBni;
  long long sCmo, sCmi, sCno, sCni;
  long long sliceA, sliceB, sliceC;  // elements per time slice
};

struct DotLayout {
  int mode;  // 0 contiguous, 1 transpose tiles, 2 trace
  int X, Y, nO;
  long long sAx, sAy, sBx, sBy;
  int O[3];
  long long sAo[3], sBo[3];
  long long sliceA, sliceB;
};

// result legs = A's free legs in order, then B's (row-major); K order is chosen to keep a
// stride-1 inner dimension for both operands when possible.  false = needs > 2 sub-dims.
bool gemm_layout(int ra, const int32_t *dA, int rb, const int32_t *dB, int c, const int8_t *pa,
                 const int8_t *pb, GemmLayout &L);

// operand-layout class of the GEMM kernels (kernels.h): 0 A[m][k] B[k][n], 1 A[m][k] B[n][k],
// 2 A[k][m] B[k][n], 3 A[k][m] B[n][k], 4 = an operand without a unit-stride inner index
int gemm_class(const GemmLayout &L);

// full contraction of A with B (rank r each, pairs (pa[i], pb[i])), or a meson trace
// (B absent: rb = 0).  false = unsupported.
bool dot_layout(int ra, const int32_t *dA, int rb, const int32_t *dB, int c, const int8_t *pa,
                const int8_t *pb, DotLayout &L);

}  // namespace micco
