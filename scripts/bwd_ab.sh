# k_prefix_bwd: parity subset, stage times, role timers (trace build in _variants/)
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "small or c4_full or c4_reduced or fused_update or hybrid_fused or rank_padding" 2>&1 | tail -2
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --stages 2>&1 >/dev/null | head -8
L=paper_conf_sc_wangwfmmd22_b200/libttemb.so; cp $L /tmp/lib_keep.so; cp _variants/libttemb_trace.so $L; touch $L
TTEMB_TRACE=1 timeout 300 python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-graph --no-pipeline 2>&1 >/dev/null | grep "trace bwd" | tail -1
cp /tmp/lib_keep.so $L; touch $L
