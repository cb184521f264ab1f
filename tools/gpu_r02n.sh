#!/bin/bash
# Mid-round GPU session: the new config benches (C5 with the tensor-core public path, C5 sharded over 2
# ranks with gloo on one GPU), and ncu --set full captures of the non-modexp kernels.
set -u
mkdir -p gpurun_out
timeout 900 python bench.py --workload c5 --no-cpu-baseline > gpurun_out/r02n_bench_c5.json 2> gpurun_out/r02n_bench_c5.err
FLB_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29541 bench.py --workload c5 --gpus 2 --steps 2 --warmup 1 \
  > gpurun_out/r02n_bench_c5_2rank_gloo.json 2> gpurun_out/r02n_bench_c5_2rank_gloo.err
timeout 1500 ncu --set full --clock-control none --import-source on \
  -k regex:"k_add|k_reduce|k_bucket|k_horner|k_pack|k_unpack|k_scan_u64|k_plan" -c 12 \
  -o gpurun_out/r02n_misc python tools/prof_misc.py > gpurun_out/r02n_ncu_misc.log 2>&1
tail -2 gpurun_out/r02n_ncu_misc.log
head -c 600 gpurun_out/r02n_bench_c5.json; echo
head -c 600 gpurun_out/r02n_bench_c5_2rank_gloo.json; echo; tail -3 gpurun_out/r02n_bench_c5_2rank_gloo.err
