python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
python tools/build_variants.py libsr_ptl4.so libsr_ptl16.so libsr_ptl2.so > /dev/null 2>&1
for L in libsr.so libsr_ptl2.so libsr_ptl4.so libsr_ptl16.so; do
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$L timeout 900 python tools/sweep.py --what pathtrace --thresholds 10,12,14 --unroll 8 --reps 3 > $O/sw_ptl_$L.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sw_ptl_$L.json'))['pathtrace']
print('$L', [(r['mode'],r['T'],round(r['ms'],2)) for r in d])"
done
for U in 6 10 12; do timeout 900 python tools/sweep.py --what pathtrace --thresholds 10,12,14 --unroll $U --reps 3 > $O/sw_ptu_$U.json 2>/dev/null; python -c "
import json;d=json.load(open('$O/sw_ptu_$U.json'))['pathtrace']
print('U=$U', [(r['mode'],r['T'],round(r['ms'],2)) for r in d])"; done
