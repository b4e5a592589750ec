#!/bin/bash
# Run under gpurun: path tracer SPEC register cap (CTAs of 128 per SM) x threshold.
TAG=${1:-ptminb}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
python tools/build_variants.py libsr_pts7.so libsr_pts8.so > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_pathtrace.py -x -q > $O/tests_$TAG.log 2>&1; tail -1 $O/tests_$TAG.log
for lib in libsr.so libsr_pts7.so libsr_pts8.so; do
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$lib timeout 600 python tools/sweep.py --what pathtrace --thresholds 8,12,16,20 --unroll 8 --reps 3 > $O/sweep_pt_${lib}_$TAG.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sweep_pt_${lib}_$TAG.json'))
print('$lib', [(r.get('mode'), r.get('T'), round(r['ms'],2)) for r in d['pathtrace']])"
done
for lib in libsr_pts7.so libsr_pts8.so; do
  echo $lib $(cuobjdump -res-usage paper_conf_cgo_damanijskymg20_b200/$lib 2>/dev/null | grep -A1 "pt_specILb0ELb1ELb1E" | grep -o "REG:[0-9]* STACK:[0-9]*")
done
rm -f paper_conf_cgo_damanijskymg20_b200/libsr_*.so
