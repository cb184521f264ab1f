# A/B of the in-tree library against a variant: bash tools/ab_variant.sh build_variants/x.so [tests...]
VAR=$1; shift
mkdir -p gpurun_out
[ $# -gt 0 ] && timeout 900 python -m pytest "$@" -q -x 2>&1 | tail -3
for lib in "" $VAR "" $VAR; do
  FLB_LIB_PATH=$lib timeout 300 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/ab.json 2>gpurun_out/ab.err || tail -5 gpurun_out/ab.err
  python -c "import json,sys; d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1]); print('${lib:-in-tree}', d['ms_per_step'], d['breakdown_ms']['t_enc'], d['breakdown_ms']['t_dec'], d['op_rates']['encrypt_per_s'], d['roofline']['frac'])"
done
