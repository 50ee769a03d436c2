set -x
mkdir -p gpurun_out/r2h
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2h/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "simulator or evict or victim" > gpurun_out/r2h/t1.log 2>&1; echo rc=$? >> gpurun_out/r2h/t1.log
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r2h/bench.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2h/launches_c5.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-c4 > gpurun_out/r2h/ncu_launch.log 2>&1
