# timing experiments of the fused kernels (TTEMB_DBG bits; results invalid)
for d in ${DBGS:-0 4}; do echo "== TTEMB_DBG=$d"; TTEMB_DBG=$d timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --stages 2>&1 >/dev/null | grep -E "fwd_prefix|bwd_rows"; done
