#!/bin/bash
# Run under gpurun: the threshold sweeps (paper Fig. 9 analogue) of every
# SPEC_LOOP workload with the current kernels, plus the ncu per-kernel pass
# (SIMT efficiency, FFMA/FFMA2 counts) of the configs[] launches.
#   bash tools/exp_sweeps.sh <tag>
TAG=${1:-r01}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
S="python tools/sweep.py --reps 3"
TS=1,2,4,8,16,24,32
timeout 900 $S --what mcml --thresholds $TS --unroll 4 > $O/sweep_mc_$TAG.json 2>/dev/null
timeout 900 $S --what mcml --thresholds $TS --unroll 1 > $O/sweep_mc_u1_$TAG.json 2>/dev/null
timeout 900 $S --what mcml --thresholds 32 --unroll 1 --defer 8 > $O/sweep_mc_defer8_$TAG.json 2>/dev/null
timeout 900 $S --what mcml --thresholds 32 --unroll 1 --defer 16 > $O/sweep_mc_defer16_$TAG.json 2>/dev/null
timeout 900 $S --what divloop --thresholds $TS > $O/sweep_dl_$TAG.json 2>/dev/null
timeout 900 $S --what rsbench --thresholds $TS > $O/sweep_rs_$TAG.json 2>/dev/null
timeout 1200 $S --what pathtrace --thresholds $TS --unroll 8 > $O/sweep_pt_$TAG.json 2>/dev/null
M=smsp__thread_inst_executed_per_inst_executed.ratio,smsp__inst_executed.sum,smsp__thread_inst_executed.sum,smsp__thread_inst_executed_pred_on.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__cycles_elapsed.avg.per_second,gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__sass_thread_inst_executed_op_ffma_pred_on.sum,sm__sass_thread_inst_executed_op_ffma2_pred_on.sum,smsp__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,launch__grid_size,launch__block_size,lts__t_bytes.sum,l1tex__t_bytes.sum
timeout 1200 ncu --metrics $M --clock-control none -k regex:"divloop|commoncall|mcml|rs_|pt_" --csv --log-file $O/simt_$TAG.csv python tools/one_launch.py > $O/simt_$TAG.log 2>&1
ls -la $O | grep $TAG
