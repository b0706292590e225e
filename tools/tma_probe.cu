// TMA layout / throughput probe for the GEMM operand staging (run on the B200 box):
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tma_probe tools/tma_probe.cu && /tmp/tma_probe
// 1. Encodes the two operand tensor maps the TMA GEMM uses (FLOAT64 elements, complex =
//    2 doubles) and checks where a box lands in shared memory:
//      K-major  X[t][row][k] (k contiguous):   smem [kq][row][k4]        dims (k4·2, row, kq, t)
//      MN-major X[t][k][row] (row contiguous): smem [kq][row/2][k4][2]   dims (2·2, k4, row/2, kq, t)
//    (non-monotonic global strides: the kq dimension steps 64 B / 4 rows).
// 2. Times back-to-back box loads on every SM (bytes/s), per layout, against a plain
//    256-byte-row box.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1); } } while (0)

static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  void *fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
  return (PFN_cuTensorMapEncodeTiled_v12000)fn;
}

__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(unsigned long long *b, unsigned cnt) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(cnt));
}
__device__ __forceinline__ void mbar_expect(unsigned long long *b, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long *b, unsigned parity) {
  asm volatile(
      "{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W;\n}\n" ::"r"(smem_u32(b)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma4(void *dst, const CUtensorMap *m, unsigned long long *bar, int c0, int c1, int c2, int c3) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];" ::"r"(
          smem_u32(dst)),
      "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void tma5(void *dst, const CUtensorMap *m, unsigned long long *bar, int c0, int c1, int c2, int c3,
                                     int c4) {
  asm volatile(
      "cp.async.bulk.tensor.5d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(
          smem_u32(dst)),
      "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4), "r"(smem_u32(bar))
      : "memory");
}

struct Maps {
  CUtensorMap kmaj, mnmaj, plain;
};

// one box of each layout into smem, copied out verbatim
__global__ void place_kernel(const __grid_constant__ Maps m, double2 *out_k, double2 *out_mn, int row0, int kq0, int t) {
  __shared__ __align__(128) double2 s[1024];
  __shared__ __align__(8) unsigned long long bar;
  if (threadIdx.x == 0) {
    mbar_init(&bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    mbar_expect(&bar, 64 * 16 * 16);
    tma4(s, &m.kmaj, &bar, 0, row0, kq0, t);
  }
  mbar_wait(&bar, 0);
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) out_k[i] = s[i];
  __syncthreads();
  if (threadIdx.x == 0) {
    mbar_expect(&bar, 64 * 16 * 16);
    tma5(s, &m.mnmaj, &bar, 0, 0, row0 / 2, kq0, t);
  }
  mbar_wait(&bar, 1);
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) out_mn[i] = s[i];
}

// throughput: each CTA streams boxes through a 4-slot ring (one thread issues, all wait)
template <int WHICH>
__global__ void stream_kernel(const __grid_constant__ Maps m, int iters, int R, int KQ, int Lt, double *sink) {
  extern __shared__ __align__(128) double2 ring[];
  __shared__ __align__(8) unsigned long long bar[4];
  if (threadIdx.x == 0) {
    for (int i = 0; i < 4; ++i) mbar_init(&bar[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](int it) {
    const int slot = it & 3;
    const int box = blockIdx.x * iters + it;
    const int t = box % Lt, kq = ((box / Lt) % (KQ / 4)) * 4, rb = ((box / Lt / (KQ / 4)) % (R / 64)) * 64;
    mbar_expect(&bar[slot], 64 * 16 * 16);
    if (WHICH == 0) tma4(ring + slot * 1024, &m.kmaj, &bar[slot], 0, rb, kq, t);
    else if (WHICH == 1) tma5(ring + slot * 1024, &m.mnmaj, &bar[slot], 0, 0, rb / 2, kq, t);
    else tma4(ring + slot * 1024, &m.plain, &bar[slot], kq * 8, rb, t, 0);
  };
  if (threadIdx.x == 0)
    for (int it = 0; it < 4 && it < iters; ++it) issue(it);
  double acc = 0;
  for (int it = 0; it < iters; ++it) {
    const int slot = it & 3;
    mbar_wait(&bar[slot], (it >> 2) & 1);
    acc += ring[slot * 1024 + threadIdx.x].x;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic reads before the next TMA write
    __syncthreads();  // the slot is free again
    if (threadIdx.x == 0 && it + 4 < iters) issue(it + 4);
  }
  if (acc == 12345.0) sink[0] = acc;
}

int main() {
  auto enc = encode_fn();
  const int Lt = 8, R = 256, K = 256;  // X[t][row][k] (K-major) and Y[t][k][row] (MN-major)
  std::vector<double2> h((size_t)Lt * R * K);
  for (int t = 0; t < Lt; ++t)
    for (int r = 0; r < R; ++r)
      for (int k = 0; k < K; ++k) h[((size_t)t * R + r) * K + k] = make_double2(t * 1e6 + r * 1e3 + k, 0.5);
  std::vector<double2> hy((size_t)Lt * R * K);
  for (int t = 0; t < Lt; ++t)
    for (int k = 0; k < K; ++k)
      for (int r = 0; r < R; ++r) hy[((size_t)t * K + k) * R + r] = make_double2(t * 1e6 + r * 1e3 + k, 0.25);
  double2 *X, *Y;
  CK(cudaMalloc(&X, h.size() * 16));
  CK(cudaMalloc(&Y, hy.size() * 16));
  CK(cudaMemcpy(X, h.data(), h.size() * 16, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(Y, hy.data(), hy.size() * 16, cudaMemcpyHostToDevice));
  Maps m;
  cuuint32_t es[5] = {1, 1, 1, 1, 1};
  {
    cuuint64_t dims[4] = {8, (cuuint64_t)R, (cuuint64_t)K / 4, (cuuint64_t)Lt};
    cuuint64_t str[3] = {(cuuint64_t)K * 16, 64, (cuuint64_t)R * K * 16};
    cuuint32_t box[4] = {8, 64, 4, 1};
    CUresult r = enc(&m.kmaj, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, X, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("encode K-major (non-monotonic strides): %d\n", (int)r);
  }
  {
    cuuint64_t dims[5] = {4, 4, (cuuint64_t)R / 2, (cuuint64_t)K / 4, (cuuint64_t)Lt};
    cuuint64_t str[4] = {(cuuint64_t)R * 16, 32, (cuuint64_t)R * 16 * 4, (cuuint64_t)R * K * 16};
    cuuint32_t box[5] = {4, 4, 32, 4, 1};
    CUresult r = enc(&m.mnmaj, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 5, Y, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("encode MN-major (non-monotonic strides): %d\n", (int)r);
  }
  {
    cuuint64_t dims[4] = {(cuuint64_t)K * 2, (cuuint64_t)R, (cuuint64_t)Lt, 1};
    cuuint64_t str[3] = {(cuuint64_t)K * 16, (cuuint64_t)R * K * 16, (cuuint64_t)R * K * 16 * Lt};
    cuuint32_t box[4] = {32, 64, 1, 1};
    CUresult r = enc(&m.plain, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, X, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("encode plain 256-B rows: %d\n", (int)r);
  }
  double2 *ok, *om;
  CK(cudaMalloc(&ok, 1024 * 16));
  CK(cudaMalloc(&om, 1024 * 16));
  const int row0 = 64, kq0 = 8, t0 = 3;
  place_kernel<<<1, 128>>>(m, ok, om, row0, kq0, t0);
  CK(cudaDeviceSynchronize());
  std::vector<double2> a(1024), b(1024);
  CK(cudaMemcpy(a.data(), ok, 1024 * 16, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(b.data(), om, 1024 * 16, cudaMemcpyDeviceToHost));
  int bad_k = 0, bad_m = 0;
  for (int kq = 0; kq < 4; ++kq)
    for (int r = 0; r < 64; ++r)
      for (int k4 = 0; k4 < 4; ++k4) {
        const double want = t0 * 1e6 + (row0 + r) * 1e3 + (kq0 + kq) * 4 + k4;
        if (a[kq * 256 + r * 4 + k4].x != want) ++bad_k;
        if (b[kq * 256 + (r >> 1) * 8 + k4 * 2 + (r & 1)].x != want) ++bad_m;
      }
  printf("placement: K-major %d bad, MN-major %d bad (of 1024)\n", bad_k, bad_m);
  printf("  K-major s[0..5].x = %.0f %.0f %.0f %.0f %.0f %.0f\n", a[0].x, a[1].x, a[2].x, a[3].x, a[4].x, a[5].x);
  printf("  MN-major s[0..5].x = %.0f %.0f %.0f %.0f %.0f %.0f\n", b[0].x, b[1].x, b[2].x, b[3].x, b[4].x, b[5].x);

  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double *sink;
  CK(cudaMalloc(&sink, 8));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int iters = 2000, smem = 4 * 1024 * 16;
  CK(cudaFuncSetAttribute(stream_kernel<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  CK(cudaFuncSetAttribute(stream_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  CK(cudaFuncSetAttribute(stream_kernel<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  const char *names[3] = {"K-major 64-B rows", "MN-major 32-B rows", "plain 256-B rows"};
  for (int w = 0; w < 3; ++w) {
    for (int ctas_per_sm : {1, 2}) {
      float best = 1e30f;
      for (int rep = 0; rep < 3; ++rep) {
        cudaEventRecord(e0);
        if (w == 0) stream_kernel<0><<<sms * ctas_per_sm, 128, smem>>>(m, iters, R, K / 4, Lt, sink);
        else if (w == 1) stream_kernel<1><<<sms * ctas_per_sm, 128, smem>>>(m, iters, R, K / 4, Lt, sink);
        else stream_kernel<2><<<sms * ctas_per_sm, 128, smem>>>(m, iters, R, K / 4, Lt, sink);
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
      }
      const double bytes = (double)sms * ctas_per_sm * iters * 16384;
      printf("%-20s ctas/SM=%d: %.1f GB/s (%.1f B/clk/SM at 1.965 GHz, L2-resident 32 MiB source)\n", names[w],
             ctas_per_sm, bytes / best * 1e-6, bytes / (best * 1e-3) / 1.965e9 / sms);
    }
  }
  return 0;
}
