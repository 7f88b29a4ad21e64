# iteration: GPU parity suite + bench with per-stage times
timeout 900 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider -x ${PYTEST_ARGS} 2>&1 | tail -25
timeout 300 python bench.py --steps 10 --warmup 3 --stages --no-e2e --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -22 gpurun_out/bench.err; cut -c1-400 gpurun_out/bench.json
