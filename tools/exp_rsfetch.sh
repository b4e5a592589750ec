#!/bin/bash
# Under gpurun: RSBench with an expensive task fetch (Fig. 9's XSBench case):
# parity, and the threshold sweep at prolog 0 / 2048 / 8192 FMAs.
TAG=${1:-x}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_rsbench.py -x -q > $O/rs_tests_$TAG.log 2>&1; tail -1 $O/rs_tests_$TAG.log
S="python tools/sweep.py --reps 5 --what rsbench --thresholds 1,2,4,8,12,16,20,24,28,32"
timeout 900 $S > $O/sweep_rs_$TAG.json 2>/dev/null
timeout 900 $S --prolog 2048 > $O/sweep_rsfetch_$TAG.json 2>/dev/null
timeout 900 $S --prolog 8192 > $O/sweep_rsfetch8k_$TAG.json 2>/dev/null
ls -la $O | grep $TAG
