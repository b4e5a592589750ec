python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k mcml > gpurun_out/exp1_tests.log 2>&1; tail -2 gpurun_out/exp1_tests.log
for L in libsr.so libsr_minb3.so; do
  SR_LIB=paper_conf_cgo_damanijskymg20_b200/$L timeout 300 python bench.py --no-cpu > gpurun_out/exp1_$L.json 2>gpurun_out/exp1_$L.err
  python -c "import json;d=json.load(open('gpurun_out/exp1_$L.json'));print('$L',d['ms_per_step'],d['pdom']['ms_per_step'],d['speedup_vs_pdom'],d['common_region_efficiency'],json.dumps(d.get('configs')))"
done
