# Timing sweep over one environment knob: VAR=<name> VALS="..." (bench c4, eager stages).
mkdir -p gpurun_out/exp
for v in $VALS; do
  env $VAR=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --stages --no-graph ${BARGS} > gpurun_out/exp/$VAR-$v.json 2> gpurun_out/exp/$VAR-$v.err
  echo "$VAR=$v $(python -c "import json; d=json.load(open('gpurun_out/exp/$VAR-$v.json')); print(round(d['ms_per_step'],4))") $(grep -E 'bwd_prefix|fwd_prefix|bwd_rows |fwd_rows ' gpurun_out/exp/$VAR-$v.err | tr -s ' ' | tr '\n' ';')"
done
