#!/bin/bash
# parity + bench + one ncu capture of the MC kernels (tag $1)
TAG=${1:-x}
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/tests_$TAG.log 2>&1; tail -2 gpurun_out/tests_$TAG.log
timeout 600 python bench.py --no-cpu > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
python -c "import json;d=json.load(open('gpurun_out/bench_$TAG.json'));print(d['ms_per_step'],d['pdom']['ms_per_step'],d['speedup_vs_pdom'],d['common_region_efficiency'], d['config']['launch'])"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:mcml -c 2 -o gpurun_out/prof_mcml_$TAG python tools/one_launch.py mcml --photons 2000000 > gpurun_out/prof_$TAG.log 2>&1
tail -1 gpurun_out/prof_$TAG.log
