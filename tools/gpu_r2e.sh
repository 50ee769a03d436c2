set -x
mkdir -p gpurun_out/r2e
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2e/build.log 2>&1
timeout 300 python tools/dbg_list.py 5 > gpurun_out/r2e/dbg5.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r2e/t1.log 2>&1; echo rc=$? >> gpurun_out/r2e/t1.log
timeout 600 python bench.py --no-c4 --no-cpu-baseline --no-e2e > gpurun_out/r2e/bench.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_plan_search --launch-skip 3 --launch-count 1 -f -o gpurun_out/r2e/prof_ks4_exh python tools/prof_search.py --mode exhaustive > gpurun_out/r2e/ncu_exh.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r2e/gpu_tests.log 2>&1; echo rc=$? >> gpurun_out/r2e/gpu_tests.log
