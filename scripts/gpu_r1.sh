set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1200 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider -x 2>&1 | tail -5
timeout 300 python bench.py --steps 20 --warmup 5 --stages --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -16 gpurun_out/bench.err; cut -c1-300 gpurun_out/bench.json
TTEMB_TRACE=1 timeout 300 python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-graph --no-pipeline 2>&1 >/dev/null | grep "trace fused" | tail -2
L=paper_conf_sc_wangwfmmd22_b200/libttemb.so; cp $L /tmp/lib_keep.so; cp _variants/libttemb_trace.so $L; touch $L
TTEMB_TRACE=1 timeout 300 python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-graph --no-pipeline 2>&1 >/dev/null | grep "trace bwd" | tail -1
cp /tmp/lib_keep.so $L; touch $L
