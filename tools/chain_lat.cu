// Micro-benchmark: issue cost of carry-chained IMAD.WIDE.U32.X sequences on sm_100a, one warp per
// SM (latency) and 4 warps per SMSP (throughput), for C independent chains interleaved.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int C>
__global__ void k_chain(uint32_t* out, uint32_t a, uint32_t b, int iters, long long* cyc) {
  uint32_t E[C][9];
#pragma unroll
  for (int c = 0; c < C; c++)
#pragma unroll
    for (int t = 0; t < 9; t++) E[c][t] = threadIdx.x + c + t;
  const long long t0 = clock64();
#pragma unroll 1
  for (int it = 0; it < iters; it++) {
    // C independent chains of 4 IMAD.WIDE.X each (8 words), written one after the other (each starts
    // with mad.lo.cc: no carry-in), so ptxas may interleave them
#pragma unroll
    for (int c = 0; c < C; c++)
#pragma unroll
      for (int j = 0; j < 8; j += 2) {
        if (j == 0)
          asm volatile("mad.lo.cc.u32 %0, %2, %3, %0;\n\tmadc.hi.cc.u32 %1, %2, %3, %1;"
                       : "+r"(E[c][j]), "+r"(E[c][j + 1]) : "r"(a + c), "r"(b));
        else
          asm volatile("madc.lo.cc.u32 %0, %2, %3, %0;\n\tmadc.hi.cc.u32 %1, %2, %3, %1;"
                       : "+r"(E[c][j]), "+r"(E[c][j + 1]) : "r"(a + c), "r"(b));
      }
  }
  const long long t1 = clock64();
  uint32_t s = 0;
#pragma unroll
  for (int c = 0; c < C; c++)
#pragma unroll
    for (int t = 0; t < 9; t++) s ^= E[c][t];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0 && blockIdx.x == 0) *cyc = t1 - t0;
}

template <int C>
void run(int warps_per_block, int blocks) {
  uint32_t* out;
  long long* cyc;
  cudaMalloc(&out, blocks * warps_per_block * 32 * 4);
  cudaMalloc(&cyc, 8);
  const int iters = 4096;
  k_chain<C><<<blocks, warps_per_block * 32>>>(out, 3, 5, iters, cyc);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  k_chain<C><<<blocks, warps_per_block * 32>>>(out, 3, 5, iters, cyc);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  long long h;
  cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  const double ops = (double)blocks * warps_per_block * 32 * iters * 4 * C;  // limb products
  printf("{\"chains\": %d, \"warps_per_sm\": %d, \"cycles_per_imad_wide_per_warp\": %.2f, "
         "\"lp_per_clk_per_sm\": %.2f}\n",
         C, warps_per_block * blocks / 148, (double)h / (iters * 4.0 * C),
         ops / (ms * 1e-3) / 148 / 1.965e9);
  cudaFree(out);
  cudaFree(cyc);
}

int main() {
  for (int w : {1, 4, 8, 16, 32}) {
    run<1>(w, 148);
    run<2>(w, 148);
    run<4>(w, 148);
  }
  run<2>(16, 2 * 148);  // 32 warps per SM as two CTAs
  run<2>(8, 8 * 148);   // 64 warps per SM
  run<4>(8, 8 * 148);
  return 0;
}
