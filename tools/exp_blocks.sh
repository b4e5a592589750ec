#!/bin/bash
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k mcml 2>&1 | tail -1
for cfg in "libsr.so 0" "libsr_t640.so 640" "libsr_t384.so 384" "libsr_t1024.so 1024" "libsr_t768.so 768"; do
  set -- $cfg
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$1 timeout 300 python bench.py --no-cpu --no-configs --steps 5 --block $2 > gpurun_out/blk_$2.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/blk_$2.json'));print('$1', $2, round(d['ms_per_step'],3), round(d['pdom']['ms_per_step'],3), d['config']['launch'])"
done
