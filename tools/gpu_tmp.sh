python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_pathtrace.py -q -x > $O/t_g20.log 2>&1; tail -1 $O/t_g20.log
timeout 900 python tools/sweep.py --what pathtrace --thresholds 12 --unroll 8 --reps 5 > $O/sw_pt20.json 2>/dev/null
python -c "
import json;d=json.load(open('$O/sw_pt20.json'))['pathtrace']
print([(r['mode'],r['T'],round(r['ms'],2)) for r in d])"
M=smsp__thread_inst_executed_per_inst_executed.ratio,smsp__inst_executed.sum,smsp__thread_inst_executed.sum,gpu__time_duration.sum
timeout 600 ncu --metrics $M --clock-control none -k regex:pt_pdom --csv --log-file $O/simt_ptpdom_g20.csv python tools/one_launch.py pathtrace --modes pdom > /dev/null 2>&1
timeout 600 ncu --section SourceCounters --clock-control none -k regex:pt_pdom -o $O/src_pt_pdom_g20 python tools/one_launch.py pathtrace --modes pdom > /dev/null 2>&1
