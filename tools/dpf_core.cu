// Feasibility probe for an FP64 limb-product path: exact 52x52 -> 104-bit products as
//   hi = fma_rd(a, b, 2^104)          (bits(hi) - bits(2^104) = floor(ab / 2^52))
//   lo = fma(a, b, (2^104 + 2^52) - hi) (bits(lo) - bits(2^52)  = ab mod 2^52)
// with the bit patterns summed into int64 column accumulators (biases removed once per column).
// Reports 52-bit limb products per clock per SM; variant ADDS selects int64 adds on the ALU pipe
// (0) or half of them as IMAD.WIDE (1).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define XL 10
template <int ADDS>
__global__ void __launch_bounds__(128) core(unsigned long long* out, double seed, int steps) {
  double a[XL], n[XL];
  unsigned long long acc[XL + 2];
#pragma unroll
  for (int j = 0; j < XL; j++) { a[j] = 4503599627370495.0 - j * 977.0 - threadIdx.x; n[j] = 4503599627370449.0 - j * 131.0; }
#pragma unroll
  for (int j = 0; j < XL + 2; j++) acc[j] = 0;
  const double C1 = 20282409603651670423947251286016.0;          // 2^104
  const double C3 = 20282409603651674927546878656512.0;          // 2^104 + 2^52
  double b = seed + threadIdx.x;
  for (int s = 0; s < steps; s++) {
#pragma unroll
    for (int j = 0; j < XL; j++) {
      double hi = __fma_rd(a[j], b, C1);
      double lo = fma(a[j], b, C3 - hi);
      if (ADDS == 0) {
        acc[j + 1] += (unsigned long long)__double_as_longlong(hi);
        acc[j] += (unsigned long long)__double_as_longlong(lo);
      } else {
        acc[j + 1] += (unsigned long long)__double_as_longlong(hi);
        unsigned long long t = (unsigned long long)__double_as_longlong(lo);
        asm volatile("mad.wide.u32 %0, %1, 1, %0;" : "+l"(acc[j]) : "r"((uint32_t)t));
        acc[j] += (t >> 32) << 32;
      }
    }
    const double m = (double)(acc[0] & 0xFFFFFFFFFFFFFull);
#pragma unroll
    for (int j = 0; j < XL; j++) {
      double hi = __fma_rd(n[j], m, C1);
      double lo = fma(n[j], m, C3 - hi);
      acc[j + 1] += (unsigned long long)__double_as_longlong(hi);
      acc[j] += (unsigned long long)__double_as_longlong(lo);
    }
#pragma unroll
    for (int j = 0; j < XL + 1; j++) acc[j] = acc[j + 1] + (j == 0 ? (acc[0] >> 52) : 0);
    acc[XL + 1] = 0;
    b = b * 0.5 + 1.0;
  }
  unsigned long long sum = 0;
#pragma unroll
  for (int j = 0; j < XL + 2; j++) sum += acc[j];
  if (sum == 12345) out[0] = sum;
}

template <int ADDS>
void run(const char* name) {
  unsigned long long* out; cudaMalloc(&out, 8);
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  int blocks = p.multiProcessorCount * 12, threads = 128, steps = 4000;
  core<ADDS><<<blocks, threads>>>(out, 3.0, 10);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float best = 1e30f;
  for (int r = 0; r < 3; r++) {
    cudaEventRecord(e0); core<ADDS><<<blocks, threads>>>(out, 3.0, steps); cudaEventRecord(e1);
    cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
  }
  double prods = (double)blocks * threads * steps * 2 * XL;
  double per_clk_sm = prods / (best * 1e-3) / (1.965e9 * p.multiProcessorCount);
  printf("{\"kind\":\"%s\",\"ms\":%.3f,\"prod52_per_clk_sm\":%.2f,\"bit2_per_clk_sm\":%.0f,\"vs_imad_wide_28\":%.2f}\n",
         name, best, per_clk_sm, per_clk_sm * 2704.0, per_clk_sm * 2704.0 / (28.0 * 1024.0));
  cudaFree(out);
}

int main() {
  run<0>("dpf_alu_adds");
  run<1>("dpf_half_imad_adds");
  return 0;
}
