python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "divloop" > $O/t_g24.log 2>&1; tail -1 $O/t_g24.log
for S in 4 8 4 8; do
  timeout 900 python tools/sweep.py --what divloop --thresholds 16 --unroll 8 --batch 64 --flags 32 --split $S --reps 10 > $O/sw_dl24_$S.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sw_dl24_$S.json'))['divloop']
print('split $S', [(r['mode'],r['T'],round(r['ms']*1000,2)) for r in d])"
done
M=smsp__thread_inst_executed_per_inst_executed.ratio,smsp__inst_executed.sum,smsp__thread_inst_executed.sum,gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__warps_active.avg.pct_of_peak_sustained_active
for S in 4 8; do
timeout 300 ncu --metrics $M --clock-control none -k regex:divloop_pool --csv python tools/one_launch.py divloop --dl-batch 64 --dl-flags 32 --dl-split $S --modes spec 2>/dev/null | grep -E "duration|issue|warps_active|ratio" | awk -F'","' '{print $(NF-2), $NF}'
done
