timeout 900 python bench.py --steps 10 --warmup 3 --stages > gpurun_out/bench1.json 2> gpurun_out/bench1.err; tail -30 gpurun_out/bench1.err; cat gpurun_out/bench1.json
