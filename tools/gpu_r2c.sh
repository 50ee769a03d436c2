set -x
mkdir -p gpurun_out/r2c
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c/build.log 2>&1
timeout 300 python tools/dbg_list.py 3 > gpurun_out/r2c/dbg3.log 2>&1
timeout 300 python tools/dbg_list.py 5 > gpurun_out/r2c/dbg5.log 2>&1
cd tests && FFS_DIST_BACKEND=gloo timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node=4 --master-addr 127.0.0.1 --master-port 29577 _dist_run.py > ../gpurun_out/r2c/dist4.log 2>&1
