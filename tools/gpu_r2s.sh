set -x
D=gpurun_out/r2s
mkdir -p $D
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $D/launches_s8.csv python tools/prof_search.py --mode bounded --slice 8 --calls 2 > $D/l.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_live|k_plan_search" --launch-skip 7 --launch-count 7 -f -o $D/prof_s8 python tools/prof_search.py --mode bounded --slice 8 --calls 2 > $D/f.log 2>&1
