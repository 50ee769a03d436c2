set -x
mkdir -p gpurun_out/r2j
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2j/build.log 2>&1
timeout 600 python tools/seg_scaling.py > gpurun_out/r2j/seg_scaling.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q > gpurun_out/r2j/t1.log 2>&1; echo rc=$? >> gpurun_out/r2j/t1.log
timeout 900 python tools/shard_emulation.py > gpurun_out/r2j/shard.log 2>&1
