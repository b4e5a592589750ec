python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 600 ncu --set full --import-source on --clock-control none -k regex:divloop -o $O/prof_dlbatch_r02d python tools/one_launch.py divloop --dl-batch 64 --modes spec > $O/p1.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:pt_spec -c 1 -o $O/prof_ptspec_r02d python tools/one_launch.py pathtrace --modes spec > $O/p2.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:rs_ -o $O/prof_rs_r02d python tools/one_launch.py rsbench > $O/p3.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:mcml_spec -c 1 -o $O/prof_mcspec_r02d python tools/one_launch.py mcml --modes spec --photons 2000000 > $O/p4.log 2>&1
ls -la $O
