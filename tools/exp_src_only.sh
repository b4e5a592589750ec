TAG=$1; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
SC="ncu --section SourceCounters --clock-control none"
OL="python tools/one_launch.py"
MCS="mcml --static --photons 131072 --iters 8"
timeout 300 $SC -k regex:divloop -o $O/src_divloop_pdom_$TAG $OL divloop --modes pdom > $O/src_log_$TAG.txt 2>&1
timeout 300 $SC -k regex:divloop -o $O/src_divloop_spec_$TAG $OL divloop --modes spec > /dev/null 2>&1
timeout 300 $SC -k regex:rs_ -o $O/src_rs_pdom_$TAG $OL rsbench --modes pdom > /dev/null 2>&1
timeout 300 $SC -k regex:rs_ -o $O/src_rs_spec_$TAG $OL rsbench --modes spec > /dev/null 2>&1
timeout 300 $SC -k regex:mcml -o $O/src_mc_pdom_$TAG $OL $MCS --modes pdom --unroll 1 > /dev/null 2>&1
timeout 300 $SC -k regex:mcml -o $O/src_mc_spec32_$TAG $OL $MCS --modes spec --threshold 32 --unroll 1 > /dev/null 2>&1
timeout 300 $SC -k regex:mcml -o $O/src_mc_spec8_$TAG $OL $MCS --modes spec --threshold 8 --unroll 1 > /dev/null 2>&1
timeout 300 $SC -k regex:mcml -o $O/src_mc_spec32u4_$TAG $OL $MCS --modes spec --threshold 32 --unroll 4 > /dev/null 2>&1
ls -la $O | grep $TAG
