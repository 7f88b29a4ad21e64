# Timing experiments on k_prefix_bwd: TTEMB_EXP bits switch parts off (results invalid).
mkdir -p gpurun_out/exp
for e in ${EXPS:-0 1 2 4 8 3 15}; do
  TTEMB_EXP=$e timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --stages --no-graph > gpurun_out/exp/e$e.json 2> gpurun_out/exp/e$e.err
  echo "EXP=$e $(grep -E 'bwd_prefix|fwd_prefix|bwd_rows ' gpurun_out/exp/e$e.err | tr -s ' ' | tr '\n' ';')"
done
