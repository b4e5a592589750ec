#!/bin/bash
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_pathtrace.py -x -q 2>&1 | tail -1
for U in 1 2 4 8; do
  python tools/sweep.py --what pathtrace --blocks 128 --thresholds 8,16,24,32 --reps 3 --unroll $U > gpurun_out/sweep_pt_u$U.json 2>/dev/null
done
python tools/sweep.py --what pathtrace --blocks 128 --thresholds 4,8,16,32 --reps 3 --flags 4 > gpurun_out/sweep_pt_coarse.json 2>/dev/null
