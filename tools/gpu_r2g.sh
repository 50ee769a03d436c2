set -x
mkdir -p gpurun_out/r2g
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2g/smoke.log 2>&1; echo smoke=$? >> gpurun_out/r2g/smoke.log
timeout 1800 python -m pytest tests -m gpu -x -q --durations=10 > gpurun_out/r2g/gpu_tests.log 2>&1; echo rc=$? >> gpurun_out/r2g/gpu_tests.log
timeout 900 python bench.py > gpurun_out/r2g/bench.log 2>&1
