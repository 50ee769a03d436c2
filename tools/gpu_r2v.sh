# REDUX warp min: parity subset, bench, slice-8 launch list + full captures of KS=3/4
set -x
D=gpurun_out/r2v
mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" > $D/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_graph.py -x -q -k "exhaustive or c5 or tiny or list or floor or every_stage or golden or C1 or C2 or graph" > $D/t.log 2>&1; echo rc=$? >> $D/t.log
timeout 900 python bench.py --no-cpu-baseline --no-c4 --no-e2e > $D/bench.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $D/launches_s8.csv python tools/prof_search.py --mode bounded --slice 8 --calls 2 > $D/l.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_live|k_plan_search" --launch-skip 7 --launch-count 7 -f -o $D/prof_s8 python tools/prof_search.py --mode bounded --slice 8 --calls 2 > $D/f.log 2>&1
