# ncu captures for the current build (run under gpurun). Args via env: KREGEX, NCU_SET
set -x
KREGEX=${KREGEX:-k_group}
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:${KREGEX} -s 6 -c ${NCU_COUNT:-2} \
  -o gpurun_out/prof python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu.log 2>&1
tail -5 gpurun_out/ncu.log
ls -la gpurun_out
