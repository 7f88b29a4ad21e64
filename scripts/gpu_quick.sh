# quick GPU check: a subset of parity tests + one bench line.  Usage: bash scripts/gpu_quick.sh tag [pytest -k expr]
tag=${1:-quick}; kexpr=${2:-"small or c4_reduced or c4_full or fused_update or pipelined or edge"}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 300 -p no:cacheprovider -x -k "$kexpr" > gpurun_out/${tag}_tests.log 2>&1
echo "tests_exit=$?" >> gpurun_out/${tag}_tests.log
tail -25 gpurun_out/${tag}_tests.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --stages > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
python -c "import json; d=json.load(open('gpurun_out/${tag}_bench.json')); print('ms/step', round(d['ms_per_step'],4), 'value', round(d['value']/1e6,1), 'M/s')"
tail -16 gpurun_out/${tag}_bench.err
