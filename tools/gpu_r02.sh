#!/bin/bash
# Run under gpurun: build, a subset (or all) of the GPU tests, one bench line.
#   bash tools/gpu_r02.sh TAG "pytest-args"   (pytest-args default: the whole -m gpu suite)
TAG=${1:-q}
SEL=${2:-tests}
python -c "import __graft_entry__ as g; g.build()"
timeout 1800 python -m pytest $SEL -m gpu -q -x > gpurun_out/tests_$TAG.log 2>&1; tail -3 gpurun_out/tests_$TAG.log
timeout 900 python bench.py --no-cpu > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -3 gpurun_out/bench_$TAG.err
python tools/bench_summary.py gpurun_out/bench_$TAG.json
