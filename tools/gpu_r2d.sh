set -x
mkdir -p gpurun_out/r2d
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2d/build.log 2>&1
timeout 300 python tools/dbg_list.py 3 > gpurun_out/r2d/dbg3.log 2>&1
timeout 300 python tools/dbg_list.py 5 > gpurun_out/r2d/dbg5.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r2d/t1.log 2>&1; echo rc=$? >> gpurun_out/r2d/t1.log
timeout 600 python bench.py --no-c4 --no-cpu-baseline --no-e2e > gpurun_out/r2d/bench.log 2>&1
