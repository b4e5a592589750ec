#!/bin/bash
# Under gpurun: path tracer tuning -- per-kernel register caps, L1 prefetch.
TAG=${1:-x}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
python tools/build_variants.py libsr_pts5.so libsr_pts7.so libsr_ptnopf.so libsr_ptp6.so > /dev/null
timeout 900 python -m pytest tests/test_gpu_pathtrace.py -x -q > $O/pt_tests_$TAG.log 2>&1; tail -1 $O/pt_tests_$TAG.log
for L in libsr.so libsr_pts5.so libsr_pts7.so libsr_ptnopf.so libsr_ptp6.so; do
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$L timeout 900 python tools/sweep.py --reps 3 --what pathtrace --thresholds 4,8 --unroll 8 > $O/sweep_pt_split_${L}_$TAG.json 2>/dev/null
done
timeout 900 python tools/sweep.py --reps 3 --what pathtrace --thresholds 8 --unroll 8 --flags 8 > $O/sweep_pt_node_$TAG.json 2>/dev/null
timeout 900 python tools/sweep.py --reps 3 --what pathtrace --thresholds 8,16 --flags 4 > $O/sweep_pt_coarse_$TAG.json 2>/dev/null
ls -la $O | grep $TAG
