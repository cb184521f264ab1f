mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_tc.py tests/test_gpu_parity.py -q -x 2>&1 | tail -2
for i in 1 2; do timeout 300 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/ab.json 2>gpurun_out/ab.err; python -c "import json,sys; d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], d['breakdown_ms']['t_enc'], d['breakdown_ms']['t_dec'], d['op_rates']['encrypt_per_s'])"; done
