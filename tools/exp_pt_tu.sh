#!/bin/bash
# Run under gpurun: path tracer threshold x merge-unroll sweep (+ MINB variants).
TAG=${1:-pttu}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
for U in 4 8 16; do
  timeout 900 python tools/sweep.py --what pathtrace --thresholds 8,12,16,20,24,32 --unroll $U --reps 3 > $O/sweep_pt_u${U}_$TAG.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sweep_pt_u${U}_$TAG.json'))
print('U=$U', [(r.get('mode'), r.get('T'), round(r['ms'],2)) for r in d['pathtrace']])"
done
python tools/build_variants.py libsr_pts5.so libsr_pts7.so libsr_ptp6.so > /dev/null 2>&1
for lib in libsr_pts5.so libsr_pts7.so libsr_ptp6.so; do
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$lib timeout 600 python tools/sweep.py --what pathtrace --thresholds 16 --unroll 8 --reps 3 > $O/sweep_pt_${lib}_$TAG.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sweep_pt_${lib}_$TAG.json'))
print('$lib', [(r.get('mode'), r.get('T'), round(r['ms'],2)) for r in d['pathtrace']])"
done
rm -f paper_conf_cgo_damanijskymg20_b200/libsr_*.so
