# c5 stage times under TTEMB_EXP variants (EXPS), rank RK (default 64)
mkdir -p gpurun_out/exp
for e in ${EXPS:-0 2048}; do
  TTEMB_EXP=$e timeout 600 python bench.py --config c5 --rank ${RK:-64} --steps 3 --warmup 2 --no-e2e --no-cpu-baseline --stages > gpurun_out/exp/c5_e$e.json 2> gpurun_out/exp/c5_e$e.err
  echo "EXP=$e $(grep -E 'bwd_rows|fwd_rows|agg |pool ' gpurun_out/exp/c5_e$e.err | tr -s ' ' | tr '\n' ';')"
done
