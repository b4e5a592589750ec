#!/bin/bash
# Run under gpurun: path tracer after the register trims (ray origin/direction kept once,
# pixel sum accumulated in the output): parity, then 8 / 9 / 10 CTAs per SM.
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_pathtrace.py -x -q > $O/tests_ptregs.log 2>&1; tail -1 $O/tests_ptregs.log
python tools/build_variants.py libsr_pt9.so libsr_pt10.so > /dev/null 2>&1
for rep in 1 2; do
for lib in libsr.so libsr_pt9.so libsr_pt10.so; do
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$lib timeout 600 python bench.py --no-cpu --steps 5 > $O/ptr_${lib}_$rep.json 2>$O/ptr_${lib}_$rep.err
  python -c "import json;d=json.load(open('$O/ptr_${lib}_$rep.json'));p=d['configs']['pathtrace'];print('$lib', round(p['pdom']['ms'],2), round(p['spec_t12']['ms'],2), p['spec_t12']['launch'])" 2>/dev/null || tail -2 $O/ptr_${lib}_$rep.err
done
done
