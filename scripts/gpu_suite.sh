# Full GPU test suite + smoke + one bench line.  Usage: bash scripts/gpu_suite.sh [tag]
tag=${1:-suite}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider -rf > gpurun_out/${tag}_tests.log 2>&1
echo "tests_exit=$?" >> gpurun_out/${tag}_tests.log
tail -15 gpurun_out/${tag}_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --stages > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
python -c "import json; d=json.load(open('gpurun_out/${tag}_bench.json')); print('ms/step', round(d['ms_per_step'],4), 'value', round(d['value']/1e6,1), 'M/s'); print(json.dumps(d['roofline'])); print(json.dumps(d['step_roofline']))"
tail -20 gpurun_out/${tag}_bench.err
