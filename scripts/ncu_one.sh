# One ncu --set full capture of the kernels matching KREGEX (run under gpurun).
KREGEX=${KREGEX:-k_tc_bwd2}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KREGEX} -s ${NCU_SKIP:-3} -c ${NCU_COUNT:-1} \
  -o gpurun_out/prof python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/ncu.log 2>&1
tail -3 gpurun_out/ncu.log
