# scratch launcher for the current gpurun experiment (see profiles/experiments.md)
python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
for L in libsr.so libsr_pttop.so libsr.so libsr_pttop.so libsr.so libsr_pttop.so; do
  SR_LIB=$PWD/paper_conf_cgo_damanijskymg20_b200/$L timeout 600 python tools/sweep.py --what pathtrace --thresholds 12 --unroll 8 --reps 7 --flags 32 > $O/sw_j_$L.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sw_j_$L.json'))['pathtrace']
print('$L pool', [(r['mode'],r['T'],round(r['ms'],2)) for r in d])"
  SR_LIB=$PWD/paper_conf_cgo_damanijskymg20_b200/$L timeout 600 python tools/sweep.py --what pathtrace --thresholds 12 --unroll 8 --reps 7 > $O/sw_j1_$L.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sw_j1_$L.json'))['pathtrace']
print('$L nopool', [(r['mode'],r['T'],round(r['ms'],2)) for r in d])"
done
SR_LIB=$PWD/paper_conf_cgo_damanijskymg20_b200/libsr_pttop.so timeout 900 python -m pytest tests/test_gpu_pathtrace.py -q > $O/t_top.log 2>&1; tail -1 $O/t_top.log
