# Round-end GPU evidence in one gpurun call: smoke, bench, GPU suite, full C3 parity, ncu launch list,
# ncu --set full of k_plan_search<4>, reference arm.  Usage: gpurun -- bash tools/gpu_evidence.sh
set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke4.log 2>&1; echo smoke=$? >> gpurun_out/smoke4.log
python bench.py > gpurun_out/bench4.log 2>&1
python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests4.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests4.log
python tests/full_parity.py 3 > gpurun_out/fp3b.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c5.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-c4 > gpurun_out/ncu_launch.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_plan_search --launch-skip 3 --launch-count 1 -f -o gpurun_out/prof_ks4_c5 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-c4 > gpurun_out/ncu_full.log 2>&1
python bench.py --impl reference > gpurun_out/bench_reference.log 2>&1
