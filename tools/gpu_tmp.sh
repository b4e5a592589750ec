python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 600 ncu --set full --import-source on --clock-control none -k regex:divloop_pool -o $O/prof_dlpool4 python tools/one_launch.py divloop --dl-batch 64 --dl-flags 32 --dl-split 4 --modes spec > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:divloop_pool -o $O/prof_dlpool1 python tools/one_launch.py divloop --dl-batch 64 --dl-flags 32 --modes spec > /dev/null 2>&1
