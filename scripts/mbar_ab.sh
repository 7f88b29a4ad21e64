L=paper_conf_sc_wangwfmmd22_b200/libttemb.so
for m in 0 1 2; do cp _variants/libttemb_m$m.so $L; touch $L; for d in 123 3 4; do echo "== mode $m DBG=$d"; TTEMB_DBG=$d timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --stages 2>&1 >/dev/null | grep -E "fwd_prefix|bwd_rows|bwd_prefix"; done; done
