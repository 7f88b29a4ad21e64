# timing experiments for the forward GEMM kernel (results invalid under TTEMB_DBG)
for d in ${DBGS:-0 1 2 4 8 15}; do
  echo "DBG=$d $(TTEMB_DBG=$d timeout 120 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --stages 2>&1 | grep -E "fwd_prefix" | head -1)"
done
