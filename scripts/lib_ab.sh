# interleaved A/B of library variants in _variants/ (LIBS), c4 graphed step + fwd/bwd rows stage times
L=paper_conf_sc_wangwfmmd22_b200/libttemb.so; cp $L /tmp/lib_keep.so
for r in $(seq ${ROUNDS:-2}); do
  for v in ${LIBS}; do
    cp _variants/$v $L; touch $L
    timeout 300 python bench.py --steps 30 --warmup 5 --no-e2e --no-cpu-baseline --stages ${BARGS} > gpurun_out/lab.json 2> gpurun_out/lab.err
    python -c "import json; d=json.load(open('gpurun_out/lab.json')); s=d['stages_us_per_step']; print('$v', round(d['ms_per_step']*1e3,1), 'us', {k: s[k] for k in (${STAGES:-'fwd_rows','bwd_rows','fwd_prefix','bwd_prefix'})})"
  done
done
cp /tmp/lib_keep.so $L; touch $L
