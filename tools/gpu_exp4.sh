#!/bin/bash
mkdir -p gpurun_out
export SQ_NVCC_EXTRA="-DSQ_TC_DEBUG=1"
python paper_conf_cluster_zhaowplw25_b200/build.py > /dev/null 2>&1 || python -c "print('build failed')"
python -c "import sys; sys.path.insert(0,'.'); import importlib.util as u; s=u.spec_from_file_location('b','paper_conf_cluster_zhaowplw25_b200/build.py'); m=u.module_from_spec(s); s.loader.exec_module(m); m.build(force=True)" > gpurun_out/e4_build.log 2>&1
timeout 300 python tools/trace_tc.py 36864 9216 4 32 > gpurun_out/e4_trace_fc1_b4.log 2>&1
timeout 300 python tools/trace_tc.py 9216 9216 4 32 > gpurun_out/e4_trace_o_b4.log 2>&1
timeout 300 python tools/trace_tc.py 36864 9216 3 32 > gpurun_out/e4_trace_fc1_b3.log 2>&1
head -70 gpurun_out/e4_trace_fc1_b4.log
