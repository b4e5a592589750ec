python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "fresnel" > $O/t_g18.log 2>&1; tail -15 $O/t_g18.log
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x -k "mcml or fullsize or full_config or outside" > $O/t_g18b.log 2>&1; tail -2 $O/t_g18b.log
for i in 1 2; do timeout 300 python bench.py --no-cpu --no-configs --steps 10 > $O/b18_$i.json 2>/dev/null; python tools/bench_summary.py $O/b18_$i.json; done
