# Role timers of k_prefix_bwd (builds a trace variant of the library on the box, then restores).
TTEMB_NVCC_FLAGS=-DTTEMB_TRACE_BUILD python -c "import __graft_entry__ as g; g._build_module().build(force=True)" > /dev/null 2>&1
TTEMB_TRACE=1 timeout 300 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-graph 2>&1 | grep 'trace bwd' | tail -1
python -c "import __graft_entry__ as g; g._build_module().build(force=True)" > /dev/null 2>&1
