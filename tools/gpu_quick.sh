#!/bin/bash
# Quick GPU iteration: the tensor-core / parity / fundamentals suites, then one default bench line.
# Outputs under gpurun_out/${TAG}_*.
set -u
TAG=${TAG:-quick}
mkdir -p gpurun_out
timeout 900 python -m pytest ${TESTS:-tests/test_gpu_tc.py tests/test_gpu_parity.py tests/test_gpu_mp.py} -q -m gpu -x 2>&1 | tail -15 > gpurun_out/${TAG}_pytest.txt
timeout 600 python bench.py --no-cpu-baseline --no-e2e ${BENCH_ARGS:-} > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
cat gpurun_out/${TAG}_pytest.txt
python - <<'PY'
import json, os
tag = os.environ.get("TAG", "quick")
try:
    d = json.load(open("gpurun_out/%s_bench.json" % tag))
    print("value %.0f ops/s  ms/step %.2f  enc %.1f ms  dec %.2f ms  frac %.3f  dec_frac %.3f" % (
        d["value"], d["ms_per_step"], d["breakdown_ms"]["t_enc"], d["breakdown_ms"]["t_dec"],
        d["roofline"]["frac"], (d.get("decrypt_roofline") or {}).get("frac", 0)))
except Exception as e:
    print("bench failed", e)
PY
tail -5 gpurun_out/${TAG}_bench.err
