set -x
D=gpurun_out/r2m
mkdir -p $D
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $D/smoke.log 2>&1; echo smoke=$? >> $D/smoke.log
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_c5_stratified.py tests/test_gpu_sanitizer.py tests/test_gpu_dag.py -x -q > $D/t.log 2>&1; echo rc=$? >> $D/t.log
timeout 900 python bench.py --no-cpu-baseline > $D/bench.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_live|k_plan_search" --launch-skip 5 --launch-count 2 -f -o $D/prof_ks4_bnd python tools/prof_search.py --mode bounded > $D/ncu_bnd.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_plan_search --launch-skip 3 --launch-count 1 -f -o $D/prof_ks4_exh python tools/prof_search.py --mode exhaustive > $D/ncu_exh.log 2>&1
