# scratch launcher for the current gpurun experiment (see profiles/experiments.md)
python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
for L in libsr.so libsr_ptl2.so libsr_ptpp8.so libsr.so libsr_ptl2.so libsr_ptpp8.so libsr.so libsr_ptl2.so libsr_ptpp8.so; do
  SR_LIB=$PWD/paper_conf_cgo_damanijskymg20_b200/$L timeout 600 python tools/sweep.py --what pathtrace --thresholds 12 --unroll 8 --reps 7 --flags 32 > $O/sw_i_$L.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sw_i_$L.json'))['pathtrace']
print('$L pool', [(r['mode'],r['T'],round(r['ms'],2)) for r in d])"
done
SR_LIB=$PWD/paper_conf_cgo_damanijskymg20_b200/libsr_ptl2.so timeout 600 ncu --metrics lts__t_sector_hit_rate.pct,dram__bytes_read.sum,gpu__time_duration.sum --clock-control none -k regex:pt_ --csv python tools/one_launch.py pathtrace --modes pdom,spec --pt-flags 32 2>/dev/null | grep -E "pt_" | cut -c1-250
