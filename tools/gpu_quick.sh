# quick: build, parity subset, bench (search legs only)
set -x
mkdir -p gpurun_out/q
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/q/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "exhaustive or c5 or tiny or list or floor or every_stage or golden or C1 or C2" > gpurun_out/q/t.log 2>&1; echo rc=$? >> gpurun_out/q/t.log
timeout 600 python bench.py --no-c4 --no-cpu-baseline --no-e2e > gpurun_out/q/bench.log 2>&1
