#!/bin/bash
# Run under gpurun: MC dynamic-claim chunk (photons a warp takes per atomic) -- the
# end-of-launch imbalance between warps is up to one chunk.  10^7 and 10^8 photons.
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
python tools/build_variants.py libsr_ch16.so libsr_ch32.so libsr_ch128.so > /dev/null 2>&1
for rep in 1 2; do
for lib in libsr.so libsr_ch16.so libsr_ch32.so libsr_ch128.so; do
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$lib timeout 300 python bench.py --no-cpu --no-configs --steps 10 > $O/ch_${lib}_$rep.json 2>/dev/null
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$lib timeout 300 python bench.py --no-cpu --no-configs --steps 3 --photons-per-gpu 100000000 > $O/ch8_${lib}_$rep.json 2>/dev/null
  python -c "import json;d=json.load(open('$O/ch_${lib}_$rep.json'));e=json.load(open('$O/ch8_${lib}_$rep.json'));print('$lib', round(d['ms_per_step'],3), round(d['pdom']['ms_per_step'],3), '1e8:', round(e['ms_per_step'],2))"
done
done
