# live grab sizes: quick parity, bench, shard emulation
set -x
D=gpurun_out/r2u
mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" > $D/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "exhaustive or c5 or tiny or list or floor or every_stage or golden or C1 or C2" > $D/t.log 2>&1; echo rc=$? >> $D/t.log
timeout 900 python bench.py --no-cpu-baseline --no-c4 --no-e2e > $D/bench.log 2>&1
timeout 900 python tools/shard_emulation.py > $D/shard.log 2>&1; cp gpurun_out/shard_emulation.json $D/
timeout 600 python tools/seg_scaling.py > $D/seg.log 2>&1
