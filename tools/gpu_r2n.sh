# bounded-mode profile after the staged k_live; full GPU suite
set -x
D=gpurun_out/r2n
mkdir -p $D
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $D/smoke.log 2>&1; echo smoke=$? >> $D/smoke.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $D/launches_bnd.csv python tools/prof_search.py --mode bounded > $D/ncu_launch.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_live|k_plan_search" --launch-skip 5 --launch-count 2 -f -o $D/prof_ks4_bnd python tools/prof_search.py --mode bounded > $D/ncu_bnd.log 2>&1
timeout 1800 python -m pytest tests -m gpu -x -q > $D/t.log 2>&1; echo rc=$? >> $D/t.log
