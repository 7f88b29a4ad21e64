for d in ${DBGS:-0 1 2 3 7}; do
  echo "DBG=$d $(TTEMB_DBG=$d TTEMB_TRACE=1 timeout 120 python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline 2>&1 | grep 'trace fused' | tail -2)"
done
