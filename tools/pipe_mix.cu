// Do IMAD.WIDE.U32.X (FMA-heavy pipe) and DFMA (FP64 pipe) co-issue?  Each thread runs NI integer
// carry chains and ND double FMA chains per iteration; we time int-only, fp64-only and mixed.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int NI, int ND>
__global__ void __launch_bounds__(256) mix(uint32_t* out, uint32_t seed, int iters) {
  uint32_t c[8];
  double d[8], e[8];
#pragma unroll
  for (int i = 0; i < 8; i++) { c[i] = seed + threadIdx.x * 7 + i; d[i] = 1.0 + 1e-9 * c[i]; e[i] = 0.999999 + 1e-12 * i; }
  uint32_t b0 = seed * 3 + 1;
  for (int it = 0; it < iters; it++) {
#pragma unroll
    for (int u = 0; u < 8; u++) {
      if (NI) asm volatile(
            "mad.lo.cc.u32 %0, %8, %8, %0; madc.hi.cc.u32 %1, %8, %8, %1;"
            "madc.lo.cc.u32 %2, %8, %1, %2; madc.hi.cc.u32 %3, %8, %1, %3;"
            "madc.lo.cc.u32 %4, %8, %3, %4; madc.hi.cc.u32 %5, %8, %3, %5;"
            "madc.lo.cc.u32 %6, %8, %5, %6; madc.hi.u32 %7, %8, %5, %7;"
            : "+r"(c[0]), "+r"(c[1]), "+r"(c[2]), "+r"(c[3]), "+r"(c[4]), "+r"(c[5]), "+r"(c[6]), "+r"(c[7])
            : "r"(b0));
      if (ND) {
#pragma unroll
        for (int i = 0; i < ND; i++) d[i] = fma(d[i], e[i], 1e-300);
      }
    }
  }
  uint32_t s = 0; double ds = 0;
#pragma unroll
  for (int i = 0; i < 8; i++) { s += c[i]; ds += d[i]; }
  if (s == 0x12345678 || ds == 1234.5) out[0] = s;
}

template <int NI, int ND>
void run(const char* name) {
  uint32_t* out; cudaMalloc(&out, 4);
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  int blocks = p.multiProcessorCount * 8, threads = 256, iters = 4000;
  mix<NI, ND><<<blocks, threads>>>(out, 1, 10);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float best = 1e30f;
  for (int r = 0; r < 3; r++) {
    cudaEventRecord(e0); mix<NI, ND><<<blocks, threads>>>(out, 1, iters); cudaEventRecord(e1);
    cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
  }
  double lanes = (double)blocks * threads * iters * 8;
  double clk = 1.965e9 * p.multiProcessorCount;
  printf("{\"kind\":\"%s\",\"ms\":%.3f,\"imad_wide_per_clk_sm\":%.2f,\"dfma_per_clk_sm\":%.2f}\n", name, best,
         NI ? lanes * 4 / (best * 1e-3) / clk : 0.0, ND ? lanes * ND / (best * 1e-3) / clk : 0.0);
  cudaFree(out);
}

int main() {
  run<1, 0>("int_only(4 IMAD.WIDE.X/u)");
  run<0, 4>("fp64_only(4 DFMA/u)");
  run<1, 4>("mixed(4 IMAD.WIDE.X + 4 DFMA /u)");
  run<1, 8>("mixed(4 IMAD.WIDE.X + 8 DFMA /u)");
  return 0;
}
