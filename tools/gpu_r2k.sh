set -x
mkdir -p gpurun_out/r2k
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2k/build.log 2>&1
timeout 600 python tools/seg_scaling.py > gpurun_out/r2k/seg_scaling.log 2>&1
