# CUDA-graph step: test, bench, shard emulation
set -x
D=gpurun_out/r2o
mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" > $D/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_graph.py -x -q > $D/t.log 2>&1; echo rc=$? >> $D/t.log
timeout 900 python bench.py --no-cpu-baseline --no-c4 > $D/bench.log 2>&1
timeout 900 python tools/shard_emulation.py > $D/shard.log 2>&1; cp gpurun_out/shard_emulation.json $D/
