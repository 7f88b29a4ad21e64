# Round evidence: parity suite, smoke, bench line, reference arm, ncu launch list (cold, serialised),
# full capture of the top kernels, optimisation breakdown.
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv,noheader
timeout 900 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider -x > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 900 python bench.py --steps 20 --warmup 5 --stages > gpurun_out/bench.json 2> gpurun_out/bench.err
tail -22 gpurun_out/bench.err; cat gpurun_out/bench.json
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; cat gpurun_out/bench_ref.json
timeout 900 python bench.py --config c5 --rank 64 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err; tail -c 300 gpurun_out/bench_c5.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -s 60 -c 40 --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-graph > /dev/null 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on \
  -k regex:"${NCU_KERNELS:-k_prefix_bwd|k_prefix_fwd|k_rows_bwd2|k_rows_fwd2|k_radix_pass|k_plan_scan|k_pool_single|k_agg_scatter|k_build_keys}" \
  -s 20 -c 12 -o gpurun_out/prof_top python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-graph > gpurun_out/ncu_top.log 2>&1
tail -2 gpurun_out/ncu_top.log
rm -rf gpurun_out/abl; ABL_CONFIGS=c4 bash scripts/ablation.sh
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --hybrid > gpurun_out/abl/c4-hybrid.json 2> gpurun_out/abl/c4-hybrid.err
