python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 1200 python -m pytest tests/test_gpu_pathtrace.py tests/test_gpu_contract.py tests/test_gpu_parity.py -q -x > $O/t_g21.log 2>&1; tail -1 $O/t_g21.log
for L in libsr.so libsr_ptbb.so; do
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$L timeout 900 python tools/sweep.py --what pathtrace --thresholds 10,12,14 --unroll 8 --reps 5 > $O/sw_pt21_$L.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sw_pt21_$L.json'))['pathtrace']
print('$L', [(r['mode'],r['T'],round(r['ms'],2)) for r in d])"
done
timeout 900 python bench.py --steps 10 --no-cpu > $O/b_g21.json 2> $O/b_g21.err; python tools/bench_summary.py $O/b_g21.json
