# Build the role-timer variant of libttemb.so into _variants/libttemb_trace.so (the in-tree
# library is rebuilt normally afterwards).  Used by scripts/bwd_ab.sh on the GPU box.
set -e
L=paper_conf_sc_wangwfmmd22_b200/libttemb.so
mkdir -p _variants
TTEMB_NVCC_FLAGS=-DTTEMB_TRACE_BUILD python -c "import sys; sys.path.insert(0, 'paper_conf_sc_wangwfmmd22_b200'); import build; build.build(force=True)"
cp $L _variants/libttemb_trace.so
python -c "import sys; sys.path.insert(0, 'paper_conf_sc_wangwfmmd22_b200'); import build; build.build(force=True)"
