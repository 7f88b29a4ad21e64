# Compare library builds that differ by nvcc defines: FLAGS_LIST="-DX=1|-DX=2" (bench c4, eager stages).
IFS='|' read -ra FL <<< "$FLAGS_LIST"
for f in "${FL[@]}"; do
  TTEMB_NVCC_FLAGS="$f" python -c "import __graft_entry__ as g; g._build_module().build(force=True)" > /dev/null 2>&1 || echo "build failed: $f"
  timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --stages > gpurun_out/eb.json 2> gpurun_out/eb.err
  echo "[$f] $(python -c "import json; d=json.load(open('gpurun_out/eb.json')); print(round(d['ms_per_step'],4))") $(grep -E 'sort_pass|unique|prefix |groups|build_keys' gpurun_out/eb.err | tr -s ' ' | tr '\n' ';')"
done
