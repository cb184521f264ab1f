#!/bin/bash
# Round-end GPU session: full parity suite, smoke, every bench line, the C2 launch list, ncu --set full
# of the three tensor-core kernels.  Outputs under gpurun_out/${TAG}_*.
set -u
TAG=${TAG:-r02final}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -q -m gpu 2>&1 | tail -5 > gpurun_out/${TAG}_pytest_gpu.txt
timeout 300 python __graft_entry__.py smoke > gpurun_out/${TAG}_smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
timeout 900 python bench.py --encrypt public --no-cpu-baseline > gpurun_out/${TAG}_bench_public.json 2> gpurun_out/${TAG}_bench_public.err
for w in c1 c3 c4 c5; do
  timeout 1200 python bench.py --workload $w --no-cpu-baseline > gpurun_out/${TAG}_bench_$w.json 2> gpurun_out/${TAG}_bench_$w.err
done
FLB_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29553 bench.py --gpus 2 --steps 2 --warmup 1 \
  > gpurun_out/${TAG}_bench2_gloo.json 2> gpurun_out/${TAG}_bench2_gloo.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${TAG}_bench_reference.json 2> gpurun_out/${TAG}_bench_reference.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e \
  > gpurun_out/${TAG}_bench_under_ncu.log 2>&1
# --set full of the three tensor-core kernels (kernel names matched on the demangled name)
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k regex:k_tc_exp_dag -c 1 -o gpurun_out/${TAG}_ncu_encrypt python tools/prof_c2.py > gpurun_out/${TAG}_ncu_encrypt.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k 'regex:k_tc_exp<.int.64>' -c 1 -o gpurun_out/${TAG}_ncu_decrypt python tools/prof_dec.py > gpurun_out/${TAG}_ncu_decrypt.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k 'regex:k_tc_exp<.int.128>' -c 1 -o gpurun_out/${TAG}_ncu_public python tools/prof_pub.py 133160 > gpurun_out/${TAG}_ncu_public.log 2>&1
# (compute-sanitizer is closed on this GPU pool: the parity suites and FLB_DEBUG_CHECKS stand in)
cat gpurun_out/${TAG}_pytest_gpu.txt gpurun_out/${TAG}_smoke.txt
for f in gpurun_out/${TAG}_bench*.json; do echo "$f"; head -c 300 "$f"; echo; done
