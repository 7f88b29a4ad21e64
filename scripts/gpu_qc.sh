# parity (GPU suite, or PYK subset) + bench stage times
timeout 900 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider -x ${PYK:+-k "$PYK"} 2>&1 | tail -4
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --stages ${BARGS} > gpurun_out/qc.json 2> gpurun_out/qc.err
python -c "import json; d=json.load(open('gpurun_out/qc.json')); print('ms/step', round(d['ms_per_step'],4), 'value', round(d['value']/1e6,1), 'M/s')"
head -14 gpurun_out/qc.err
