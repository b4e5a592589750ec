python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_pathtrace.py -q -k schedule > $O/t_g13.log 2>&1; tail -3 $O/t_g13.log
