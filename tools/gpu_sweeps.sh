#!/bin/bash
# Run under gpurun: the threshold sweeps (Fig. 9 analogue) of every SPEC_LOOP workload
# with the current kernels -> gpurun_out/sweep_*_$TAG.json (tools/sweep_report.py).
TAG=${1:-r02}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
S="python tools/sweep.py --reps 3"
TS=1,2,4,8,12,16,20,24,32
timeout 900 $S --what mcml --thresholds $TS --unroll 4 > $O/sweep_mc_$TAG.json 2>/dev/null
timeout 900 $S --what divloop --thresholds $TS --unroll 8 > $O/sweep_dl_$TAG.json 2>/dev/null
timeout 900 $S --what divloop --thresholds $TS --unroll 8 --batch 64 > $O/sweep_dlbatch_$TAG.json 2>/dev/null
timeout 900 $S --what rsbench --thresholds $TS --unroll 12 > $O/sweep_rs_$TAG.json 2>/dev/null
timeout 900 $S --what rsbench --thresholds $TS --prolog 2048 --unroll 12 > $O/sweep_rsfetch_$TAG.json 2>/dev/null
timeout 1500 $S --what pathtrace --thresholds $TS --unroll 8 > $O/sweep_pt_$TAG.json 2>/dev/null
timeout 1500 $S --what pathtrace --thresholds 1,4,8,16,24,32 --flags 4 > $O/sweep_ptcoarse_$TAG.json 2>/dev/null
timeout 1500 $S --what pathtrace --thresholds $TS --unroll 8 --flags 32 > $O/sweep_ptpool_$TAG.json 2>/dev/null
ls -la $O/sweep_*_$TAG.json
