#!/bin/bash
# Run under gpurun: bench + ncu evidence for one round. Usage: tools/gpu_profile.sh <tag>
set -x
TAG=${1:-r01}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err
M=smsp__thread_inst_executed_per_inst_executed.ratio,smsp__inst_executed.sum,smsp__thread_inst_executed.sum,smsp__thread_inst_executed_pred_on.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__cycles_elapsed.avg.per_second,gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__sass_thread_inst_executed_op_ffma_pred_on.sum,smsp__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,launch__grid_size,launch__block_size
timeout 900 ncu --metrics $M --clock-control none -k regex:"divloop|commoncall|mcml" --csv --log-file $O/simt_$TAG.csv python tools/one_launch.py > $O/simt_$TAG.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv python bench.py --steps 2 --warmup 1 --no-cpu --no-configs > $O/launches_$TAG.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:mcml_spec -c 1 -o $O/prof_mcml_spec_$TAG python tools/one_launch.py mcml --modes spec > $O/prof_$TAG.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:mcml_pdom -c 1 -o $O/prof_mcml_pdom_$TAG python tools/one_launch.py mcml --modes pdom >> $O/prof_$TAG.log 2>&1
ls -la $O
