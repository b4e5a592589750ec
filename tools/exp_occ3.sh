#!/bin/bash
# Run under gpurun: MCML occupancy variants after the div_dom/sqrt_dom step
# (fewer live registers): 2 x 640 (default) vs 3 x 512 / 3 x 480 at 40 registers.
TAG=${1:-occ3}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
python tools/build_variants.py libsr_t512m3.so libsr_t480m3.so > /dev/null 2>&1
for rep in 1 2; do
for lib in libsr.so libsr_t512m3.so libsr_t480m3.so; do
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$lib timeout 300 python bench.py --no-cpu --no-configs --steps 10 > $O/occ3_${lib}_$rep.json 2>$O/occ3_${lib}_$rep.err
  python -c "import json;d=json.load(open('$O/occ3_${lib}_$rep.json'));print('$lib', round(d['ms_per_step'],3), round(d['pdom']['ms_per_step'],3), d['config']['launch'])" 2>/dev/null || tail -2 $O/occ3_${lib}_$rep.err
done
done
