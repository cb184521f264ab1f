// flb_inst.cu — explicit instantiation of the run_* launchers (and so of their kernels) for one
// (X, T) frame split.  build.py compiles this file once per split with
// -DFLB_INST_X=<X> -DFLB_INST_T=<T> -DFLB_INST_ENC=<0|1> -DFLB_INST_DEC=<0|1>, in parallel; the
// C ABI in flb_api.cu refers to these instantiations through the extern declarations in flb_core.cuh.
#define FLB_INST_TU 1
#include "flb_core.cuh"

#if FLB_INST_ENC
FLB_ENC_DECLS(, FLB_INST_X, FLB_INST_T)
#endif
#if FLB_INST_DEC
FLB_DEC_DECLS(, FLB_INST_X, FLB_INST_T)
#endif
#if defined(FLB_INST_TC)
FLB_TC_DECLS(, FLB_INST_TC)
#if FLB_INST_TC == 64
FLB_TC_DAG_DECLS()
#endif
#endif

#if defined(FLB_INST_TC) && (FLB_INST_TC == 64 || FLB_INST_TC == 128) && FLB_TC_PROF
#if FLB_INST_TC == 128
#define flb_debug_tc_prof flb_debug_tc_prof128  // the k_tc_exp<128> object's own counters
#endif
// profiling builds only (FLB_NVCC_EXTRA=-DFLB_TC_PROF=1; not in include/): per-phase cycle totals of
// thread 0 of the 2048-bit tensor-core Montgomery kernel (tools/tc_phases.py)
extern "C" int flb_debug_tc_prof(uint64_t* out16, int reset) {
  unsigned long long h[16];
  FLB_CK(cudaMemcpyFromSymbol(h, flb::tc::g_tc_prof, sizeof(h)));
  for (int i = 0; i < 16; i++) out16[i] = h[i];
  if (reset) {
    unsigned long long z[16] = {};
    FLB_CK(cudaMemcpyToSymbol(flb::tc::g_tc_prof, z, sizeof(z)));
  }
  return FLB_OK;
}
#endif
