#!/bin/bash
# GPU A/B of library variants: the tensor-core parity suites on the in-tree build, then tools/ab_tc.py
# (key-holder encryption + decryption) and tools/ab_pub.py (public encryption) for the in-tree build
# and every build_variants/<name>.so named in VARIANTS.  Outputs under gpurun_out/${TAG}_*.
set -u
TAG=${TAG:-ab}
mkdir -p gpurun_out
timeout 900 python -m pytest ${TESTS:-tests/test_gpu_tc.py tests/test_gpu_tc_wide.py} -q -m gpu -x 2>&1 | tail -15 > gpurun_out/${TAG}_pytest.txt
cat gpurun_out/${TAG}_pytest.txt
for v in main ${VARIANTS:-}; do
  if [ "$v" = main ]; then lib=""; else lib=build_variants/$v.so; fi
  FLB_LIB_PATH=$lib timeout 600 python tools/ab_tc.py 2>&1 | tail -1 | tee -a gpurun_out/${TAG}_ab_tc.jsonl
  if [ -n "${PUB:-1}" ]; then
    FLB_LIB_PATH=$lib timeout 600 python tools/ab_pub.py 2>&1 | tail -1 | tee -a gpurun_out/${TAG}_ab_pub.jsonl
  fi
done
