# Run under gpurun: the driver's round-end checks on the current tree (GPU tests incl. the bounds-checked build, smoke, one bench line)
python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > $O/final2_tests.log 2>&1; tail -3 $O/final2_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/final2_smoke.log 2>&1; tail -1 $O/final2_smoke.log
timeout 900 python bench.py --steps 5 --warmup 3 > $O/final2_bench.json 2> $O/final2_bench.err; tail -c 200 $O/final2_bench.json
