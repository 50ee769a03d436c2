set -x
mkdir -p gpurun_out/r2f
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2f/build.log 2>&1
./tools/issue_bench > gpurun_out/r2f/issue_bench.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_live|k_plan_search" --launch-skip 5 --launch-count 2 -f -o gpurun_out/r2f/prof_bnd python tools/prof_search.py --mode bounded > gpurun_out/r2f/ncu_bnd.log 2>&1
timeout 900 python tools/shard_emulation.py > gpurun_out/r2f/shard.log 2>&1
timeout 900 python bench.py > gpurun_out/r2f/bench.log 2>&1
