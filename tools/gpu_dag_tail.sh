set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_tc.py tests/test_gpu_tc_wide.py -q -m gpu -x 2>&1 | tail -3
for c in 133160 132608 66580; do timeout 300 python tools/ab_tc.py 2048 $c 2>&1 | tail -1; done
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k 'regex:k_tc_exp<.int.64>' -c 1 -o gpurun_out/r02final_ncu_decrypt python tools/prof_dec.py > gpurun_out/r02final_ncu_decrypt.log 2>&1
tail -1 gpurun_out/r02final_ncu_decrypt.log
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k 'regex:k_tc_exp<.int.128>' -c 1 -o gpurun_out/r02final_ncu_public python tools/prof_pub.py 133160 > gpurun_out/r02final_ncu_public.log 2>&1
tail -1 gpurun_out/r02final_ncu_public.log
