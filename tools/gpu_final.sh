#!/bin/bash
# Round-end GPU session: full parity suite, smoke, every bench line, the C2 launch list, ncu --set full
# of the three tensor-core kernels, compute-sanitizer.  Outputs under gpurun_out/${TAG}_*.
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
i=0
for name in encrypt decrypt; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tc_exp --launch-skip $i -c 1 \
    -o gpurun_out/${TAG}_ncu_$name python tools/prof_c2.py > gpurun_out/${TAG}_ncu_$name.log 2>&1
  i=$((i + 1))
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tc_exp -c 1 \
  -o gpurun_out/${TAG}_ncu_public python tools/prof_pub.py 133160 > gpurun_out/${TAG}_ncu_public.log 2>&1
{
  for tool in memcheck racecheck synccheck initcheck; do
    echo "-- $tool (small)"; timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_small.py 2>&1 | tail -3
  done
  for tool in memcheck synccheck; do
    echo "-- $tool (dag, 20000 elements)"; timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_small.py dag 2>&1 | tail -3
  done
} > gpurun_out/${TAG}_sanitizers.txt 2>&1
cat gpurun_out/${TAG}_pytest_gpu.txt gpurun_out/${TAG}_smoke.txt gpurun_out/${TAG}_sanitizers.txt
for f in gpurun_out/${TAG}_bench*.json; do echo "$f"; head -c 300 "$f"; echo; done
