// Probe: exact u8 x u8 -> s32 GEMM on the 5th-gen tensor cores (tcgen05.mma kind::i8, TMEM
// accumulator), hand-written PTX, no-swizzle K-major core-matrix layouts.  D[128 x N] = A[128 x K]
// * B[N x K]^T, checked element by element against a host reference.  Also times back-to-back
// MMAs.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/tc_i8_probe tools/tc_i8_probe.cu
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d: %s\n", #x, __LINE__, cudaGetErrorString(e)); exit(1); } } while (0)

constexpr int M = 128, K = 256, N = 256;

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// byte offset of element (row, k) in a K-major no-swizzle core-matrix layout with `kchunks` 16-byte
// chunks per row: core matrix = 8 rows x 16 B (128 B contiguous), K chunks adjacent (LBO = 128 B),
// 8-row groups SBO = kchunks * 128 B apart
__host__ __device__ __forceinline__ uint32_t cm_off(uint32_t row, uint32_t k, uint32_t kchunks) {
  return (row >> 3) * (kchunks * 128u) + (k >> 4) * 128u + (row & 7u) * 16u + (k & 15u);
}

__device__ __forceinline__ uint64_t make_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr & 0x3FFFFu) >> 4);
  d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
  d |= (uint64_t)1 << 46;  // version 1 (sm_100)
  return d;                // base offset 0, lbo mode 0, layout SWIZZLE_NONE (0)
}

__device__ __forceinline__ uint32_t idesc_i8(int m, int n) {
  return (2u << 4) /* S32 accum */ | (0u << 7) /* A u8 */ | (0u << 10) /* B u8 */ |
         ((uint32_t)(n >> 3) << 17) | ((uint32_t)(m >> 4) << 24);
}

__global__ void __launch_bounds__(128, 1) probe(const uint8_t* __restrict__ A, const uint8_t* __restrict__ B,
                                                int32_t* __restrict__ D, int reps, long long* cycles) {
  extern __shared__ __align__(1024) uint8_t smem[];
  uint8_t* sA = smem;                 // M x K
  uint8_t* sB = smem + M * K;         // N x K
  __shared__ __align__(8) uint64_t mbar;
  __shared__ uint32_t tmem_base_sh;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  constexpr uint32_t kch = K / 16;
  for (int i = tid; i < M * K; i += blockDim.x) sA[cm_off(i / K, i % K, kch)] = A[i];
  for (int i = tid; i < N * K; i += blockDim.x) sB[cm_off(i / K, i % K, kch)] = B[i];
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&mbar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" :: "r"(smem_u32(&tmem_base_sh)), "n"(256));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_base_sh;
  const uint32_t idesc = idesc_i8(M, N);
  long long t0 = clock64();
  uint32_t phase = 0;
  for (int r = 0; r < reps; r++) {
    if (tid == 0) {
#pragma unroll
      for (int ks = 0; ks < K / 32; ks++) {
        const uint64_t ad = make_desc(smem_u32(sA) + ks * 2 * 128, 128, kch * 128);
        const uint64_t bd = make_desc(smem_u32(sB) + ks * 2 * 128, 128, kch * 128);
        const uint32_t acc = ks > 0 ? 1u : 0u;
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}"
            :: "r"(tmem), "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
      }
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(smem_u32(&mbar)));
    }
    // wait for the MMAs
    asm volatile(
        "{\n\t.reg .pred P1;\n\tWAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra WAIT_%=;\n\t}" :: "r"(smem_u32(&mbar)), "r"(phase));
    phase ^= 1;
    asm volatile("tcgen05.fence::after_thread_sync;");
  }
  long long t1 = clock64();
  if (tid == 0) cycles[0] = t1 - t0;
  // TMEM -> registers -> global: warp w reads lanes 32w..32w+31 (rows), 32 columns at a time
  for (int c0 = 0; c0 < N; c0 += 32) {
    uint32_t v[32];
    const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)c0;
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
          "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
          "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    const int row = warp * 32 + lane;
#pragma unroll
    for (int j = 0; j < 32; j++) D[row * N + c0 + j] = (int32_t)v[j];
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(tmem), "n"(256));
}

int main() {
  std::vector<uint8_t> A(M * K), B(N * K);
  srand(12345);
  for (auto& x : A) x = (uint8_t)(rand() & 0xFF);
  for (auto& x : B) x = (uint8_t)(rand() & 0xFF);
  // make a few rows/cols extreme
  for (int k = 0; k < K; k++) { A[k] = 0xFF; B[k] = 0xFF; }
  uint8_t *dA, *dB; int32_t* dD; long long* dc;
  CK(cudaMalloc(&dA, M * K)); CK(cudaMalloc(&dB, N * K)); CK(cudaMalloc(&dD, M * N * 4)); CK(cudaMalloc(&dc, 8));
  CK(cudaMemcpy(dA, A.data(), M * K, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dB, B.data(), N * K, cudaMemcpyHostToDevice));
  const int smem = M * K + N * K;
  CK(cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  for (int reps : {1, 1000}) {
    CK(cudaMemset(dD, 0, M * N * 4));
    probe<<<1, 128, smem>>>(dA, dB, dD, reps, dc);
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
    std::vector<int32_t> D(M * N);
    long long cyc;
    CK(cudaMemcpy(D.data(), dD, M * N * 4, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(&cyc, dc, 8, cudaMemcpyDeviceToHost));
    long bad = 0;
    for (int m = 0; m < M; m++)
      for (int n = 0; n < N; n++) {
        int64_t s = 0;
        for (int k = 0; k < K; k++) s += (int64_t)A[m * K + k] * B[n * K + k];
        if (s != D[m * N + n]) { if (bad < 5) printf("mismatch m=%d n=%d got %d want %lld\n", m, n, D[m * N + n], (long long)s); bad++; }
      }
    const double macs = (double)reps * M * N * K;
    printf("{\"reps\": %d, \"mismatches\": %ld, \"cycles\": %lld, \"macs_per_cycle_per_sm\": %.1f}\n", reps, bad, cyc,
           macs / (double)cyc);
  }
  return 0;
}
