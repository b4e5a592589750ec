python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -x > $O/t_g15.log 2>&1; tail -2 $O/t_g15.log
