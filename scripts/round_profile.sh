# Round evidence: bench line, ncu launch list (cold, serialised), full capture of the top kernels.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv,noheader
timeout 900 python bench.py --steps 20 --warmup 5 --stages > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -s 60 -c 24 --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_tc_bwd2|k_tc_p|k_rows_bwd|k_rows_fwd" -s 8 -c 4 \
  -o gpurun_out/prof_top python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_top.log 2>&1
tail -2 gpurun_out/ncu_top.log
