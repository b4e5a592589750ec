# scratch launcher: the bounds-checked build over every kernel variant
python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_bounds.py -q > $O/t_bounds.log 2>&1; tail -3 $O/t_bounds.log
SR_LIB=$PWD/paper_conf_cgo_damanijskymg20_b200/libsr_bounds.so timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_pathtrace.py tests/test_gpu_rsbench.py -q -x > $O/t_bounds_parity.log 2>&1; tail -2 $O/t_bounds_parity.log
