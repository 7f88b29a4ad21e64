# e2e leg vs HostStepPipeline depth (c4)
for d in ${DEPTHS:-2 3 4}; do
  timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-depth $d 2>/dev/null > gpurun_out/e2e_d$d.json
  python - "$d" <<'PY'
import json, sys
d = json.loads(open(f"gpurun_out/e2e_d{sys.argv[1]}.json").readline())
print("depth", sys.argv[1], "e2e ms", round(d["e2e"]["ms_per_step"], 3), "dev ms", round(d["ms_per_step"], 4))
PY
done
