#!/bin/bash
# Window-size sweep of the tensor-core paths (FLB_WMAX = largest sliding window of the schedules):
# tools/ab_tc.py timings and the DRAM bytes of one k_tc_exp_dag launch per setting, then one
# ncu --set full capture of k_tc_exp_dag at the default.  Outputs under gpurun_out/${TAG}_*.
set -u
TAG=${TAG:-wmax}
mkdir -p gpurun_out
for w in ${WMAXES:-7 5 4}; do
  FLB_WMAX=$w timeout 600 python tools/ab_tc.py 2>&1 | tail -1 | sed "s/^{/{\"wmax\": $w, /" | tee -a gpurun_out/${TAG}_ab_tc.jsonl
  FLB_WMAX=$w timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
    --clock-control none --kernel-name-base demangled -k regex:k_tc_exp_dag -c 1 --csv \
    python tools/prof_dec.py 133160 > gpurun_out/${TAG}_dram_w$w.csv 2>&1
  grep -E "dram__bytes|gpu__time" gpurun_out/${TAG}_dram_w$w.csv | cut -c1-400
done
if [ -n "${FULL:-1}" ]; then
  timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k regex:k_tc_exp_dag -c 1 -o gpurun_out/${TAG}_ncu_dag python tools/prof_dec.py 133160 > gpurun_out/${TAG}_ncu_dag.log 2>&1
  tail -2 gpurun_out/${TAG}_ncu_dag.log
fi
