#!/bin/bash
# One GPU session: parity tests, smoke, bench (1 GPU), 2-rank gloo bench on the same GPU,
# ncu launch list and one full ncu capture of the encrypt kernel.  Outputs under gpurun_out/.
set -u
TAG=${TAG:-run}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu 2>&1 | tail -4 > gpurun_out/${TAG}_pytest_gpu.txt
timeout 300 python __graft_entry__.py smoke > gpurun_out/${TAG}_smoke.txt 2>&1
timeout 900 python bench.py ${BENCH_ARGS:-} > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
if [ "${MULTI:-1}" = "1" ]; then
  FLB_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
    --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 1 --no-e2e \
    > gpurun_out/${TAG}_bench2_gloo.json 2> gpurun_out/${TAG}_bench2_gloo.err
fi
if [ "${NCU:-1}" = "1" ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e \
    > gpurun_out/${TAG}_bench_under_ncu.log 2>&1
  # the tensor-core kernels of the step: key-holder stage 1 (k_tc_exp<32>), stage 2 and decryption (k_tc_exp<64>)
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"${NCU_K:-k_tc_exp}" -c ${NCU_C:-3} \
    -o gpurun_out/${TAG}_prof_enc python tools/prof_c2.py > gpurun_out/${TAG}_ncu_full.log 2>&1
fi
cat gpurun_out/${TAG}_pytest_gpu.txt gpurun_out/${TAG}_smoke.txt
tail -c 3000 gpurun_out/${TAG}_bench.json
tail -c 600 gpurun_out/${TAG}_bench2_gloo.json 2>/dev/null; tail -3 gpurun_out/${TAG}_bench2_gloo.err 2>/dev/null
