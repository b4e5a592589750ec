# scratch launcher for the current gpurun experiment: profile + the path-tracer sweeps
TAG=${1:-r02n}
bash tools/gpu_profile.sh $TAG
O=gpurun_out
S="python tools/sweep.py --reps 3"
TS=1,2,4,8,12,16,20,24,32
timeout 1500 $S --what pathtrace --thresholds $TS --unroll 8 > $O/sweep_pt_$TAG.json 2>/dev/null
timeout 1500 $S --what pathtrace --thresholds 1,4,8,16,24,32 --flags 4 > $O/sweep_ptcoarse_$TAG.json 2>/dev/null
timeout 1500 $S --what pathtrace --thresholds $TS --unroll 8 --flags 32 > $O/sweep_ptpool_$TAG.json 2>/dev/null
ls -la $O/sweep_*_$TAG.json
