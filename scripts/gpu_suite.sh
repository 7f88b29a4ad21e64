# Full GPU test suite + smoke + one bench line.
timeout 900 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider -x 2>&1 | tail -4
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --stages > gpurun_out/qc.json 2> gpurun_out/qc.err
python -c "import json; d=json.load(open('gpurun_out/qc.json')); print('ms/step', round(d['ms_per_step'],4), 'value', round(d['value']/1e6,1), 'M/s')"
