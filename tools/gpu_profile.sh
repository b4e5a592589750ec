#!/bin/bash
# Run under gpurun: GPU tests, bench, and the ncu evidence for one round.
#   bash tools/gpu_profile.sh <tag> [quick]
# Outputs under gpurun_out/ (summarised into profiles/ by tools/summarize_ncu.py).
set -x
TAG=${1:-r01}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
# SASS hashes of the kernels this run measures (tools/summarize_ncu.py stores them with the
# measurements, so a later local rebuild cannot be mistaken for the measured code)
python -c "import json,sys; sys.path.insert(0,'tools'); import sass_regions as S; json.dump(S.kernel_hashes('divloop_|commoncall_|mcml_|pt_|rs_'), open('$O/sass_hashes_$TAG.json','w'))"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/gpu_$TAG.txt
if [ "$2" != "quick" ]; then
  timeout 1200 python -m pytest tests -m gpu -q > $O/tests_$TAG.log 2>&1; tail -3 $O/tests_$TAG.log
  timeout 300 python __graft_entry__.py smoke > $O/smoke_$TAG.log 2>&1; tail -1 $O/smoke_$TAG.log
fi
timeout 900 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err
M=smsp__thread_inst_executed_per_inst_executed.ratio,smsp__inst_executed.sum,smsp__thread_inst_executed.sum,smsp__thread_inst_executed_pred_on.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__cycles_elapsed.avg.per_second,gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__sass_thread_inst_executed_op_ffma_pred_on.sum,sm__sass_thread_inst_executed_op_ffma2_pred_on.sum,smsp__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,launch__grid_size,launch__block_size,lts__t_bytes.sum,l1tex__t_bytes.sum
# every kernel family at its configs[] size (bench launch configuration)
timeout 1200 ncu --metrics $M --clock-control none -k regex:"divloop|commoncall|mcml|rs_|pt_" --csv --log-file $O/simt_$TAG.csv python tools/one_launch.py > $O/simt_$TAG.log 2>&1
# the batched-prolog divloop kernels and the static-assignment RSBench kernel
timeout 600 ncu --metrics $M --clock-control none -k regex:divloop --csv --log-file $O/simt_dlbatch_$TAG.csv python tools/one_launch.py divloop --dl-batch 64 > /dev/null 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:rs_ --csv --log-file $O/simt_rsstatic_$TAG.csv python tools/one_launch.py rsbench --modes spec --rs-flags 2 > /dev/null 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:divloop --csv --log-file $O/simt_dlpool_$TAG.csv python tools/one_launch.py divloop --dl-batch 64 --dl-flags 32 --modes spec > /dev/null 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:divloop --csv --log-file $O/simt_dlpool4_$TAG.csv python tools/one_launch.py divloop --dl-batch 64 --dl-flags 32 --dl-split 4 --modes spec > /dev/null 2>&1
timeout 900 ncu --metrics $M --clock-control none -k regex:pt_spec --csv --log-file $O/simt_ptpool_$TAG.csv python tools/one_launch.py pathtrace --modes spec --pt-flags 32 > /dev/null 2>&1
# the simulator validation launches (static assignment, the oracle replays every warp)
timeout 600 ncu --metrics $M --clock-control none -k regex:mcml --csv --log-file $O/simt_mcstatic_$TAG.csv python tools/one_launch.py mcml --static --photons 131072 --iters 8 --modes pdom,spec --threshold 32 --unroll 1 > /dev/null 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:mcml --csv --log-file $O/simt_mcstatic8_$TAG.csv python tools/one_launch.py mcml --static --photons 131072 --iters 8 --modes spec --threshold 8 --unroll 1 > /dev/null 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:mcml --csv --log-file $O/simt_mcstaticu4_$TAG.csv python tools/one_launch.py mcml --static --photons 131072 --iters 8 --modes spec --threshold 32 --unroll 4 > /dev/null 2>&1
# per-instruction SourceCounters of the simulator-validation launches (tools/region_check.py)
SC="ncu --section SourceCounters --clock-control none"
OL="python tools/one_launch.py"
MCS="mcml --static --photons 131072 --iters 8"
timeout 300 $SC -k regex:divloop -o $O/src_divloop_pdom_$TAG $OL divloop --modes pdom > /dev/null 2>&1
timeout 300 $SC -k regex:divloop -o $O/src_divloop_spec_$TAG $OL divloop --modes spec > /dev/null 2>&1
timeout 300 $SC -k regex:rs_ -o $O/src_rs_pdom_$TAG $OL rsbench --modes pdom > /dev/null 2>&1
timeout 300 $SC -k regex:rs_ -o $O/src_rs_spec_$TAG $OL rsbench --modes spec > /dev/null 2>&1
timeout 300 $SC -k regex:mcml -o $O/src_mc_pdom_$TAG $OL $MCS --modes pdom --unroll 1 > /dev/null 2>&1
timeout 300 $SC -k regex:mcml -o $O/src_mc_spec32_$TAG $OL $MCS --modes spec --threshold 32 --unroll 1 > /dev/null 2>&1
timeout 300 $SC -k regex:mcml -o $O/src_mc_spec8_$TAG $OL $MCS --modes spec --threshold 8 --unroll 1 > /dev/null 2>&1
timeout 300 $SC -k regex:mcml -o $O/src_mc_spec32u4_$TAG $OL $MCS --modes spec --threshold 32 --unroll 4 > /dev/null 2>&1
timeout 300 $SC -k regex:divloop_pool -o $O/src_dlpool_$TAG $OL divloop --dl-batch 64 --dl-flags 32 --modes spec > /dev/null 2>&1
timeout 300 $SC -k regex:divloop_pool -o $O/src_dlpool4_$TAG $OL divloop --dl-batch 64 --dl-flags 32 --dl-split 4 --modes spec > /dev/null 2>&1
timeout 600 $SC -k regex:pt_pdom -o $O/src_pt_pdom_$TAG $OL pathtrace --modes pdom > /dev/null 2>&1
timeout 600 $SC -k regex:pt_spec -o $O/src_pt_spec_$TAG $OL pathtrace --modes spec > /dev/null 2>&1
timeout 600 $SC -k regex:pt_spec -o $O/src_pt_pool_$TAG $OL pathtrace --modes spec --pt-flags 32 > /dev/null 2>&1
# full captures of the path tracer kernels (PDOM and the default split merge)
# (one kernel per process: a second full capture in the same process came back mostly NaN)
timeout 900 ncu --set full --import-source on --clock-control none -k regex:pt_pdom -c 1 -o $O/prof_ptpdom_$TAG $OL pathtrace --modes pdom > $O/prof_pt_$TAG.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:pt_spec -c 1 -o $O/prof_ptspec_$TAG $OL pathtrace --modes spec >> $O/prof_pt_$TAG.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:pt_spec -c 1 -o $O/prof_ptpool_$TAG $OL pathtrace --modes spec --pt-flags 32 >> $O/prof_pt_$TAG.log 2>&1
# launch list of one short bench run (shares, not absolutes)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv python bench.py --steps 2 --warmup 1 --no-cpu --no-configs > $O/launches_$TAG.log 2>&1
# full captures of the dominant kernel (and its PDOM baseline), at 2M photons
timeout 900 ncu --set full --import-source on --clock-control none -k regex:mcml -c 2 -o $O/prof_mcml_$TAG python tools/one_launch.py mcml --photons 2000000 > $O/prof_$TAG.log 2>&1
# dram traffic of the bench-sized dominant kernel
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:mcml_spec -c 1 --csv --log-file $O/traffic_$TAG.csv python tools/one_launch.py mcml --modes spec > /dev/null 2>&1
ls -la $O | tail -30
# configs[4] at N = 1: the full 10^9 photons on one GPU (3 timed steps)
timeout 900 python bench.py --photons-per-gpu 1000000000 --steps 3 --warmup 3 --no-configs --no-cpu > $O/bench_c5_$TAG.json 2> $O/bench_c5_$TAG.err
# CPU baselines of every config, one core and all host cores
timeout 900 python tools/cpu_baselines.py --out $O/cpu_baselines_$TAG.json > /dev/null 2> $O/cpu_baselines_$TAG.err
# the reports compress ~5x; gpurun brings back at most 64 MiB (gunzip them here)
gzip -f $O/*_$TAG.ncu-rep
du -sh $O
