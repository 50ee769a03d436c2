# round-2 GPU call B: bounded-mode live-mask compaction -- parity, bench, ncu
set -x
mkdir -p gpurun_out/r2b
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2b/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "list or exhaustive or c5 or tiny or every_stage or golden or C1 or C2 or shard" > gpurun_out/r2b/t1.log 2>&1; echo rc=$? >> gpurun_out/r2b/t1.log
timeout 600 python bench.py --no-c4 --no-cpu-baseline > gpurun_out/r2b/bench.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_live|k_plan_search" --launch-skip 5 --launch-count 2 -f -o gpurun_out/r2b/prof_bnd python tools/prof_search.py --mode bounded > gpurun_out/r2b/ncu_bnd.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r2b/gpu_tests.log 2>&1; echo rc=$? >> gpurun_out/r2b/gpu_tests.log
