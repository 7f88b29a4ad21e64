set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
nproc
timeout 1200 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider 2>&1 | tail -40
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -5
timeout 900 python bench.py --steps 5 --warmup 3 --stages --no-cpu-baseline > gpurun_out/bench1.json 2> gpurun_out/bench1.err; tail -30 gpurun_out/bench1.err; cat gpurun_out/bench1.json
