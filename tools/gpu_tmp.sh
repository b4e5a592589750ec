python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k divloop_pool > $O/t_g14.log 2>&1; tail -1 $O/t_g14.log
timeout 600 python tools/sweep.py --what divloop --thresholds 16 --unroll 8 --batch 64 --flags 32 --split 4 --reps 10 > $O/sw_dl_g14.json 2>/dev/null
python -c "
import json
d=json.load(open('$O/sw_dl_g14.json'))['divloop']
print('split4 cta pool', [(r['mode'],r['T'],round(r['ms']*1000,1), round(r['region_eff'],3)) for r in d])"
python tools/build_variants.py libsr_ptnopf.so > /dev/null 2>&1
for L in libsr.so libsr_ptnopf.so; do
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$L timeout 900 python tools/sweep.py --what pathtrace --thresholds 8,12,16 --unroll 8 --reps 5 > $O/sw_pt14_$L.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sw_pt14_$L.json'))['pathtrace']
print('$L', [(r['mode'],r['T'],round(r['ms'],2)) for r in d])"
done
