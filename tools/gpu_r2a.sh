# round-2 GPU call A: suite, bench, ncu of the exhaustive and bounded KS = 4 kernels
set -x
mkdir -p gpurun_out/r2a
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2a/smoke.log 2>&1; echo smoke=$? >> gpurun_out/r2a/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q --durations=15 > gpurun_out/r2a/gpu_tests.log 2>&1; echo rc=$? >> gpurun_out/r2a/gpu_tests.log
timeout 900 python bench.py > gpurun_out/r2a/bench.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_plan_search --launch-skip 3 --launch-count 1 -f -o gpurun_out/r2a/prof_ks4_exh python tools/prof_search.py --mode exhaustive > gpurun_out/r2a/ncu_exh.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_plan_search --launch-skip 3 --launch-count 1 -f -o gpurun_out/r2a/prof_ks4_bnd python tools/prof_search.py --mode bounded > gpurun_out/r2a/ncu_bnd.log 2>&1
