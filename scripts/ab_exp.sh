# interleaved A/B of the default path vs TTEMB_EXP=$B_EXP (graph step time, c4), ROUNDS rounds
for r in $(seq ${ROUNDS:-4}); do
  for e in 0 ${B_EXP}; do
    TTEMB_EXP=$e timeout 300 python bench.py --steps 30 --warmup 5 --no-e2e --no-cpu-baseline ${BARGS} 2>/dev/null > gpurun_out/ab.json
    python -c "import json; d=json.load(open('gpurun_out/ab.json')); print('EXP=$e', round(d['ms_per_step']*1e3,1), 'us')"
  done
done
