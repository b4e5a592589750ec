python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k divloop_pool > $O/t_g17.log 2>&1; tail -1 $O/t_g17.log
M=smsp__thread_inst_executed_per_inst_executed.ratio,smsp__inst_executed.sum,smsp__thread_inst_executed.sum,gpu__time_duration.sum
timeout 300 ncu --metrics $M --clock-control none -k regex:divloop --csv --log-file $O/simt_dlpool_g17.csv python tools/one_launch.py divloop --dl-batch 64 --dl-flags 32 --modes spec > /dev/null 2>&1
grep -E "ratio|duration" $O/simt_dlpool_g17.csv | cut -d, -f5,13-16
