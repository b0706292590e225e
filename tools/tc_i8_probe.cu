// tc_i8_probe.cu — hardware probe for the tcgen05 kind::i8 building blocks used by the
// Ozaki-scheme FP64 emulation: smem descriptors for K-major
// SWIZZLE_NONE operands in two core-matrix orders, the instruction descriptor, TMEM
// accumulator layout (row m = lane m, column n = column n) and throughput for N = 32..256.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o build/tc_i8_probe tools/tc_i8_probe.cu
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e_), __LINE__); exit(1); } } while (0)

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t sdesc(uint32_t addr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((addr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= 1ULL << 46;  // version 1 (sm_100)
  return d;         // base offset 0, lbo mode 0, layout SWIZZLE_NONE (0)
}

__host__ __device__ constexpr uint32_t idesc_i8(int M, int N) {
  return (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

__device__ __forceinline__ void mma_i8(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
               "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}\n"
               :: "r"(d), "l"(a), "l"(b), "r"(idesc), "r"(acc));
}

__device__ __forceinline__ void mbar_init(uint64_t *b, int n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(b)), "r"(n));
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity) {
  asm volatile("{\n\t.reg .pred p;\n\tWAIT_%=:\n\t"
               "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
               "@!p bra WAIT_%=;\n\t}\n" :: "r"(smem_u32(b)), "r"(parity));
}
__device__ __forceinline__ void mma_commit(uint64_t *b) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(smem_u32(b)));
}

// canonical K-major SWIZZLE_NONE tile: R rows x KB bytes; core matrix (rg, kc) = 8 rows x 16 B.
// order 0: [rg][kc] (LBO = 128, SBO = KB/16*128); order 1: [kc][rg] (LBO = R/8*128, SBO = 128)
__device__ __forceinline__ int core_off(int r, int k, int R, int KB, int order) {
  int rg = r >> 3, kc = k >> 4;
  int core = order == 0 ? rg * (KB / 16) + kc : kc * (R / 8) + rg;
  return core * 128 + (r & 7) * 16 + (k & 15);
}

template <int N>
__global__ void probe_kernel(const int8_t *A, const int8_t *B, int *D, int KB, int order, int reps) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint32_t tmem_base;
  __shared__ __align__(8) uint64_t bar;
  const int M = 128;
  int8_t *As = (int8_t *)sm;
  int8_t *Bs = (int8_t *)sm + M * KB;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  for (int i = tid; i < M * KB; i += blockDim.x) { int r = i / KB, k = i % KB; As[core_off(r, k, M, KB, order)] = A[i]; }
  for (int i = tid; i < N * KB; i += blockDim.x) { int r = i / KB, k = i % KB; Bs[core_off(r, k, N, KB, order)] = B[i]; }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" :: "r"(smem_u32(&tmem_base)), "n"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) mbar_init(&bar, 1);
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tm = tmem_base;
  const uint32_t lboA = order == 0 ? 128 : (M / 8) * 128, sboA = order == 0 ? (KB / 16) * 128 : 128;
  const uint32_t lboB = order == 0 ? 128 : (N / 8) * 128, sboB = order == 0 ? (KB / 16) * 128 : 128;
  const uint32_t stepA = order == 0 ? 256 : 2 * lboA, stepB = order == 0 ? 256 : 2 * lboB;
  long long t0 = 0, t1 = 0;
  if (warp == 0 && lane == 0) {
    t0 = clock64();
    for (int r = 0; r < reps; ++r)
      for (int ks = 0; ks < KB / 32; ++ks)
        mma_i8(tm, sdesc(smem_u32(As) + ks * stepA, lboA, sboA), sdesc(smem_u32(Bs) + ks * stepB, lboB, sboB),
               idesc_i8(M, N), (r | ks) ? 1u : 0u);
    mma_commit(&bar);
  }
  mbar_wait(&bar, 0);
  if (warp == 0 && lane == 0) t1 = clock64();
  asm volatile("tcgen05.fence::after_thread_sync;");
  // warp w reads lanes 32w..32w+31; 32x32b.x8: 8 consecutive columns per thread
  for (int c = 0; c < N; c += 8) {
    uint32_t v[8];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
                 : "r"(tm + ((uint32_t)(warp * 32) << 16) + c));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    for (int j = 0; j < 8; ++j) D[(warp * 32 + lane) * N + c + j] = (int)v[j];
  }
  if (warp == 0 && lane == 0) D[M * N] = (int)(t1 - t0);
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(tm), "n"(512));
}

template <int N>
void run(int KB, int order, int reps) {
  const int M = 128;
  std::vector<int8_t> a(M * KB), b(N * KB);
  srand(1234 + N + order);
  for (auto &x : a) x = (int8_t)(rand() % 256 - 128);
  for (auto &x : b) x = (int8_t)(rand() % 256 - 128);
  int8_t *dA, *dB; int *dD;
  CK(cudaMalloc(&dA, a.size())); CK(cudaMalloc(&dB, b.size())); CK(cudaMalloc(&dD, (M * N + 1) * 4));
  CK(cudaMemcpy(dA, a.data(), a.size(), cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dB, b.data(), b.size(), cudaMemcpyHostToDevice));
  const int smem = (M + N) * KB;
  CK(cudaFuncSetAttribute(probe_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  probe_kernel<N><<<1, 128, smem>>>(dA, dB, dD, KB, order, reps);
  CK(cudaGetLastError());
  CK(cudaDeviceSynchronize());
  std::vector<int> d(M * N + 1);
  CK(cudaMemcpy(d.data(), dD, d.size() * 4, cudaMemcpyDeviceToHost));
  int bad = 0;
  for (int m = 0; m < M; ++m)
    for (int n = 0; n < N; ++n) {
      long long s = 0;
      for (int k = 0; k < KB; ++k) s += (int)a[m * KB + k] * (int)b[n * KB + k];
      s *= reps;
      if (s != d[m * N + n]) { if (bad < 3) printf("  mismatch m=%d n=%d got %d want %lld\n", m, n, d[m * N + n], s); ++bad; }
    }
  double macs = (double)M * N * KB * reps;
  printf("N=%d KB=%d order=%d reps=%d: %s (%d bad); %d cycles, %.0f MAC/clk\n", N, KB, order, reps,
         bad ? "FAIL" : "ok", bad, d[M * N], macs / d[M * N]);
  cudaFree(dA); cudaFree(dB); cudaFree(dD);
}

// throughput with NACC independent accumulators (columns NACC*N <= 512), issue only
template <int N, int NACC>
__global__ void thr_kernel(int *out, int KB, int reps) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint32_t tmem_base;
  __shared__ __align__(8) uint64_t bar;
  const int M = 128;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  for (int i = tid; i < (M + N) * KB; i += blockDim.x) sm[i] = (uint8_t)(i * 7);
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" :: "r"(smem_u32(&tmem_base)), "n"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) mbar_init(&bar, 1);
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tm = tmem_base;
  const uint8_t *As = sm, *Bs = sm + M * KB;
  const uint32_t lboA = (M / 8) * 128, lboB = (N / 8) * 128;
  if (warp == 0 && lane == 0) {
    long long t0 = clock64();
    for (int r = 0; r < reps; ++r)
      for (int ks = 0; ks < KB / 32; ++ks)
#pragma unroll
        for (int q = 0; q < NACC; ++q)
          mma_i8(tm + q * N, sdesc(smem_u32(As) + ks * 2 * lboA, lboA, 128), sdesc(smem_u32(Bs) + ks * 2 * lboB, lboB, 128),
                 idesc_i8(M, N), (r | ks) ? 1u : 0u);
    mma_commit(&bar);
    mbar_wait(&bar, 0);
    long long t1 = clock64();
    double macs = (double)M * N * KB * reps * NACC;
    printf("thr N=%d NACC=%d: %.0f MAC/clk (%.1f cycles/MMA)\n", N, NACC, macs / (t1 - t0), (double)(t1 - t0) / (reps * (KB / 32) * NACC));
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(tm), "n"(512));
}

template <int N, int NACC>
void thr() {
  const int KB = 128, smem = (128 + N) * KB;
  CK(cudaFuncSetAttribute(thr_kernel<N, NACC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  thr_kernel<N, NACC><<<1, 128, smem>>>(nullptr, KB, 64);
  CK(cudaDeviceSynchronize());
}

int main() {
  thr<32, 1>(); thr<32, 6>(); thr<32, 12>();
  thr<64, 1>(); thr<64, 2>(); thr<64, 4>(); thr<64, 6>(); thr<64, 8>();
  thr<80, 6>(); thr<96, 5>();
  thr<128, 1>(); thr<128, 2>(); thr<128, 4>();
  thr<256, 1>(); thr<256, 2>();

  for (int order = 0; order < 2; ++order) {
    run<64>(64, order, 1);
    run<32>(128, order, 1);
  }
  run<16>(64, 1, 1);
  run<128>(64, 1, 1);
  run<256>(64, 1, 1);
  for (int reps : {64, 256}) {
    run<32>(128, 1, reps);
    run<64>(128, 1, reps);
    run<128>(128, 1, reps);
    run<256>(128, 1, reps);
  }
  return 0;
}
