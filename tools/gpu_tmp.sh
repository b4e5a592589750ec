python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
python tools/build_variants.py libsr_pt8.so libsr_pt7.so libsr_pt10.so > /dev/null 2>&1
S="python tools/sweep.py --what pathtrace --reps 3"
for U in 2 3 4 6; do timeout 900 $S --thresholds 8,10,12,14 --unroll $U > $O/sw_pt6_u$U.json 2>/dev/null; done
for L in libsr_pt8.so libsr_pt7.so libsr_pt10.so; do SR_LIB=paper_conf_cgo_damanijskymg20_b200/$L timeout 900 $S --thresholds 10,12 --unroll 4 > $O/sw_pt6_$L.json 2>/dev/null; done
for f in $O/sw_pt6_*.json; do python -c "
import json;d=json.load(open('$f'))['pathtrace']
print('$f'.split('/')[-1], [(r['mode'],r['T'],round(r['ms'],2), round(r.get('region_eff',0),3)) for r in d])"; done
