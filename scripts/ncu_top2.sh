# Full ncu capture of the current top kernels (one launch each, after warm-up), plus SASS-level source.
mkdir -p gpurun_out
timeout 1500 ncu --set full --clock-control none --import-source on \
  -k regex:"${NCU_KERNELS:-k_prefix_bwd|k_prefix_fwd|k_rows_fwd2|k_pool|k_build_keys|k_scan}" -s ${NCU_SKIP:-16} -c ${NCU_COUNT:-8} \
  -o gpurun_out/prof_top2 python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-graph > gpurun_out/ncu_top2.log 2>&1
tail -3 gpurun_out/ncu_top2.log
