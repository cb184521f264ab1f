#!/bin/bash
# Refresh the bench lines after late changes: TC parity suites, then the default, public and C1 bench
# lines.  Outputs under gpurun_out/${TAG}_*.
set -u
TAG=${TAG:-refresh}
mkdir -p gpurun_out
timeout 900 python -m pytest ${TESTS:-tests/test_gpu_tc.py tests/test_gpu_tc_wide.py tests/test_gpu_parity.py tests/test_gpu_host_pipeline.py} -q -m gpu -x 2>&1 | tail -3
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
timeout 900 python bench.py --encrypt public --no-cpu-baseline > gpurun_out/${TAG}_bench_public.json 2> gpurun_out/${TAG}_bench_public.err
for w in ${WORKLOADS:-c1}; do
  timeout 1200 python bench.py --workload $w --no-cpu-baseline > gpurun_out/${TAG}_bench_$w.json 2> gpurun_out/${TAG}_bench_$w.err
done
for f in gpurun_out/${TAG}_bench*.json; do echo "$f"; head -c 400 "$f"; echo; done
