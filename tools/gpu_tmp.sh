# scratch launcher: the driver's round-end checks on the current tree
python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > $O/final_tests.log 2>&1; tail -3 $O/final_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/final_smoke.log 2>&1; tail -1 $O/final_smoke.log
timeout 900 python bench.py > $O/final_bench.json 2> $O/final_bench.err; tail -c 400 $O/final_bench.json
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $O/final_ref.json 2> $O/final_ref.err; tail -c 300 $O/final_ref.json
