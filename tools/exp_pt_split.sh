#!/bin/bash
# Under gpurun: parity of the split-leaf path tracer, its threshold / unroll
# sweep, and full ncu captures of the node-merge and split kernels.
TAG=${1:-x}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_pathtrace.py -x -q > $O/pt_tests_$TAG.log 2>&1; tail -1 $O/pt_tests_$TAG.log
S="python tools/sweep.py --reps 3 --what pathtrace"
timeout 900 $S --thresholds 4,8,16,24,32 --unroll 8 --flags 8 > $O/sweep_pt_split_$TAG.json 2>/dev/null
timeout 900 $S --thresholds 8,16 --unroll 4 --flags 8 > $O/sweep_pt_split_u4_$TAG.json 2>/dev/null
timeout 900 $S --thresholds 8,16 --unroll 16 --flags 8 > $O/sweep_pt_split_u16_$TAG.json 2>/dev/null
timeout 900 ncu --set full --import-source on --clock-control none -k regex:pt_spec -c 1 -o $O/prof_pt_node_$TAG python tools/one_launch.py pathtrace --modes spec > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:pt_spec -c 1 -o $O/prof_pt_split_$TAG python tools/one_launch.py pathtrace --modes spec --pt-flags 8 > /dev/null 2>&1
ls -la $O | grep $TAG
