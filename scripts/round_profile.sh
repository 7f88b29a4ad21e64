# Round evidence: parity suite, smoke, bench line, ncu launch list (cold, serialised), full capture of the top kernels.
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv,noheader
timeout 900 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider -x > gpurun_out/pytest_gpu.log 2>&1; tail -5 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 900 python bench.py --steps 20 --warmup 5 --stages > gpurun_out/bench.json 2> gpurun_out/bench.err
tail -30 gpurun_out/bench.err; cat gpurun_out/bench.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -s 60 -c 40 --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"${NCU_KERNELS:-k_tc_bwd2|k_tc_fwd|k_rows_bwd2|k_rows_fwd2|k_agg_scatter|k_radix_pass}" -s 12 -c 6 \
  -o gpurun_out/prof_top python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-graph > gpurun_out/ncu_top.log 2>&1
tail -2 gpurun_out/ncu_top.log
