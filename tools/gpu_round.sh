#!/bin/bash
# Round-end style GPU session: parity suite, smoke, every bench config, the C2 launch list, and one
# ncu --set full capture per tensor-core kernel of the C2 step (encryption, decryption; one
# process each).  Outputs under gpurun_out/${TAG}_*.
set -u
TAG=${TAG:-round}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -q -m gpu 2>&1 | tail -4 > gpurun_out/${TAG}_pytest_gpu.txt
timeout 300 python __graft_entry__.py smoke > gpurun_out/${TAG}_smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
for w in c1 c3 c4 c5; do
  timeout 900 python bench.py --workload $w --no-cpu-baseline > gpurun_out/${TAG}_bench_$w.json 2> gpurun_out/${TAG}_bench_$w.err
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e \
  > gpurun_out/${TAG}_bench_under_ncu.log 2>&1
# prof_c2.py launches the key-holder encryption (k_tc_exp_dag: both stages, one launch) first, then
# the decryption (k_tc_exp<64>); FLB_TC_DAG=0 gives the two-launch form (stage 1, stage 2, decryption)
i=0
for name in encrypt decrypt; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tc_exp --launch-skip $i -c 1 \
    -o gpurun_out/${TAG}_ncu_$name python tools/prof_c2.py > gpurun_out/${TAG}_ncu_$name.log 2>&1
  i=$((i + 1))
done
cat gpurun_out/${TAG}_pytest_gpu.txt gpurun_out/${TAG}_smoke.txt
for f in gpurun_out/${TAG}_bench*.json; do echo "$f"; head -c 400 "$f"; echo; done
