#!/bin/bash
# Run under gpurun: MCML CTA-size / register-cap variants (bench headline + PDOM).
TAG=${1:-occ2}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
python tools/build_variants.py libsr_t576.so libsr_t640.so libsr_t704.so libsr_t416m3.so > /dev/null 2>&1
for rep in 1 2; do
for lib in libsr.so libsr_t576.so libsr_t640.so libsr_t416m3.so libsr_t704.so; do
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$lib timeout 300 python bench.py --no-cpu --no-configs --steps 10 > $O/occ2_${lib}_$rep.json 2>$O/occ2_${lib}_$rep.err
  python -c "import json;d=json.load(open('$O/occ2_${lib}_$rep.json'));print('$lib', round(d['ms_per_step'],3), round(d['pdom']['ms_per_step'],3), d['config']['launch'])" 2>/dev/null || tail -2 $O/occ2_${lib}_$rep.err
done
done
