# ncu --set full of the fused kernels (one launch each) + a quick bench line.  Usage: bash scripts/ncu_tt.sh tag
tag=${1:-tt}
mkdir -p gpurun_out
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --stages > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
python -c "import json; d=json.load(open('gpurun_out/${tag}_bench.json')); print('ms/step', round(d['ms_per_step'],4), 'value', round(d['value']/1e6,1), 'M/s')"
tail -14 gpurun_out/${tag}_bench.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"${KREGEX:-k_tt|k_prefix_bwd}" -s ${NCU_SKIP:-6} -c ${NCU_COUNT:-3} \
  -o gpurun_out/${tag} python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-graph --no-pipeline > gpurun_out/${tag}_ncu.log 2>&1
tail -3 gpurun_out/${tag}_ncu.log
