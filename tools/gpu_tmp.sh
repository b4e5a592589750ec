# scratch launcher for the current gpurun experiment (see profiles/experiments.md)
python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
for L in libsr.so libsr_ptcs.so libsr_ptpw.so libsr_ptcspw.so libsr.so libsr_ptcs.so libsr_ptpw.so libsr_ptcspw.so; do
  SR_LIB=$PWD/paper_conf_cgo_damanijskymg20_b200/$L timeout 600 python tools/sweep.py --what pathtrace --thresholds 12 --unroll 8 --reps 7 --flags 32 > $O/sw_w_$L.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sw_w_$L.json'))['pathtrace']
print('$L', [(r['mode'],r['T'],round(r['ms'],2)) for r in d])"
done
for L in libsr_ptcspw.so libsr_ptpw.so; do
SR_LIB=$PWD/paper_conf_cgo_damanijskymg20_b200/$L timeout 900 python -m pytest tests/test_gpu_pathtrace.py -q -k "pool or full_config or small" > $O/t_$L.log 2>&1; tail -1 $O/t_$L.log
done
