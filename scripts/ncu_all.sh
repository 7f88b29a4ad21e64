# full ncu set for every kernel of one bench step (skip warm-up launches)
set -x
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_|ttemb" -s ${NCU_SKIP:-100} -c ${NCU_COUNT:-40} \
  -o gpurun_out/prof_all python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_all.log 2>&1
tail -3 gpurun_out/ncu_all.log
