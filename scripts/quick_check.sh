# Quick GPU check after a kernel change: parity subset + stage timings.
timeout 600 python -m pytest tests/test_gpu_parity.py -q --timeout 300 -p no:cacheprovider -x ${PYK:+-k "$PYK"} 2>&1 | tail -3
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --stages ${BARGS} > gpurun_out/qc.json 2> gpurun_out/qc.err
python -c "import json; d=json.load(open('gpurun_out/qc.json')); print('ms/step', round(d['ms_per_step'],4), 'value', round(d['value']/1e6,1), 'M/s')"
head -12 gpurun_out/qc.err
