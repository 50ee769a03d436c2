set -x
mkdir -p gpurun_out/r2l
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2l/smoke.log 2>&1; echo smoke=$? >> gpurun_out/r2l/smoke.log
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2l/gpu_tests.log 2>&1; echo rc=$? >> gpurun_out/r2l/gpu_tests.log
timeout 900 python bench.py > gpurun_out/r2l/bench.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_plan_search --launch-skip 3 --launch-count 1 -f -o gpurun_out/r2l/prof_ks4_exh python tools/prof_search.py --mode exhaustive > gpurun_out/r2l/ncu_exh.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_live|k_plan_search" --launch-skip 5 --launch-count 2 -f -o gpurun_out/r2l/prof_bnd python tools/prof_search.py --mode bounded > gpurun_out/r2l/ncu_bnd.log 2>&1
