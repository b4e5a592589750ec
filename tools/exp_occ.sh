#!/bin/bash
# Run under gpurun: occupancy variants of the MC and path-tracer kernels.
TAG=${1:-occ}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
python tools/build_variants.py libsr_t640.so libsr_t384.so libsr_t768.so libsr_pts7.so > /dev/null 2>&1
for cfg in "libsr.so 0" "libsr_t384.so 384" "libsr_t640.so 640" "libsr_t768.so 768"; do
  set -- $cfg
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$1 timeout 300 python bench.py --no-cpu --no-configs --steps 5 --block $2 > $O/occ_$2_$TAG.json 2>/dev/null
  python -c "import json;d=json.load(open('$O/occ_$2_$TAG.json'));print('$1', $2, round(d['ms_per_step'],3), round(d['pdom']['ms_per_step'],3), d['config']['launch'])"
done
for lib in libsr.so libsr_pts7.so; do
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$lib timeout 600 python tools/sweep.py --what pathtrace --thresholds 4,8 --unroll 8 --reps 3 > $O/occ_pt_${lib}_$TAG.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/occ_pt_${lib}_$TAG.json'))
for r in d['pathtrace']: print('$lib', r.get('mode'), r.get('T'), round(r['ms'],2))"
done
cuobjdump -res-usage paper_conf_cgo_damanijskymg20_b200/libsr_t384.so 2>/dev/null | grep -A1 mcml_spec | grep -o "REG:[0-9]*" | head -2
