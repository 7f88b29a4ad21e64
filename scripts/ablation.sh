# ablation switches + the paper-design comparator on the bench workload (c4), one GPU.
mkdir -p gpurun_out/abl
[ -n "$ABL_TESTS" ] && timeout 900 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider -x > gpurun_out/abl/pytest_gpu.log 2>&1
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline"
for cfgn in ${ABL_CONFIGS:-c4 c3}; do
  timeout 300 $B --config $cfgn > gpurun_out/abl/$cfgn-base.json 2> gpurun_out/abl/$cfgn-base.err
  timeout 300 $B --config $cfgn --no-reuse > gpurun_out/abl/$cfgn-no_reuse.json 2> gpurun_out/abl/$cfgn-no_reuse.err
  timeout 300 $B --config $cfgn --no-agg > gpurun_out/abl/$cfgn-no_agg.json 2> gpurun_out/abl/$cfgn-no_agg.err
  timeout 300 $B --config $cfgn --unfused > gpurun_out/abl/$cfgn-unfused.json 2> gpurun_out/abl/$cfgn-unfused.err
  timeout 300 $B --config $cfgn --ids perm > gpurun_out/abl/$cfgn-perm.json 2> gpurun_out/abl/$cfgn-perm.err
  timeout 300 $B --config $cfgn --ids perm --bijection 16 > gpurun_out/abl/$cfgn-perm_bij.json 2> gpurun_out/abl/$cfgn-perm_bij.err
  timeout 600 python bench.py --impl paper --config $cfgn --steps 5 --warmup 3 > gpurun_out/abl/$cfgn-paper.json 2> gpurun_out/abl/$cfgn-paper.err
done
for f in gpurun_out/abl/*.json; do echo "$f $(python -c "import json,sys; d=json.load(open('$f')); print(round(d['ms_per_step'],3), 'ms', round(d['value']/1e6,1), 'M/s')" 2>&1 | tail -1)"; done
