# scratch launcher for the current gpurun experiment (see profiles/experiments.md)
python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
for L in libsr.so libsr_ptflat.so libsr_pttile.so libsr_pttf.so libsr.so libsr_pttf.so; do
  SR_LIB=$PWD/paper_conf_cgo_damanijskymg20_b200/$L timeout 600 python tools/sweep.py --what pathtrace --thresholds 12 --unroll 8 --reps 7 --flags 32 > $O/sw_v_$L.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sw_v_$L.json'))['pathtrace']
print('$L', [(r['mode'],r['T'],round(r['ms'],2)) for r in d])"
done
for L in libsr_pttile.so libsr_pttf.so; do
  SR_LIB=$PWD/paper_conf_cgo_damanijskymg20_b200/$L timeout 600 python tools/sweep.py --what pathtrace --thresholds 8,12,16 --unroll 8 --reps 5 > $O/sw_v1_$L.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sw_v1_$L.json'))['pathtrace']
print('nopool $L', [(r['mode'],r['T'],round(r['ms'],2)) for r in d])"
done
SR_LIB=$PWD/paper_conf_cgo_damanijskymg20_b200/libsr_pttf.so timeout 900 python -m pytest tests/test_gpu_pathtrace.py -q -k "bit_exact or brute or full_config" > $O/t_tf.log 2>&1; tail -3 $O/t_tf.log
