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
