# Bench lines for the other BASELINE configs (parity for all of them is in tests/test_gpu_parity.py).
mkdir -p gpurun_out/sweep
for c in c1 c2 c3 c4; do
  timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/sweep/$c.json 2>/dev/null
done
for r in 32 64 128; do
  timeout 600 python bench.py --config c5 --rank $r --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/sweep/c5-r$r.json 2>/dev/null
done
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --opt adagrad > gpurun_out/sweep/c4-adagrad.json 2>/dev/null
for f in gpurun_out/sweep/*.json; do python -c "
import json,sys; d=json.load(open('$f')); print('$f', d['config']['workload'], round(d['ms_per_step'],4), 'ms', round(d['value']/1e6,1), 'M/s', 'e2e', round(d['e2e']['value']/1e6,1) if d.get('e2e') else None)" 2>&1 | tail -1; done
