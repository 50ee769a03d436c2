# Round-2 GPU evidence in one gpurun call: smoke, GPU suite, bench (+ reference arm),
# ncu launch list, ncu --set full of the exhaustive KS=4 kernel, the bounded KS=4 pair
# (k_live + list search) and the fused C4 step, shard emulation, segment scaling, issue
# microbenchmark.   gpurun --timeout 4000 -- bash tools/gpu_evidence_r2.sh
set -x
D=${D:-gpurun_out/ev2}
mkdir -p $D
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $D/smoke.log 2>&1; echo smoke=$? >> $D/smoke.log
timeout 1800 python -m pytest tests -m gpu -q --durations=15 > $D/gpu_tests.log 2>&1; echo rc=$? >> $D/gpu_tests.log
timeout 900 python bench.py > $D/bench.log 2>&1
timeout 900 python bench.py --impl reference > $D/bench_reference.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $D/launches_c5.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-c4 > $D/ncu_launch.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_plan_search --launch-skip 3 --launch-count 1 -f -o $D/prof_ks4_exh python tools/prof_search.py --mode exhaustive > $D/ncu_exh.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_live|k_plan_search" --launch-skip 5 --launch-count 2 -f -o $D/prof_ks4_bnd python tools/prof_search.py --mode bounded > $D/ncu_bnd.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_evict_ticks" --launch-skip 3 --launch-count 1 -f -o $D/prof_c4 python -c "
import sys; sys.path.insert(0, '.')
import bench, torch
from paper_conf_hpdc_hui0s25_b200 import ffs
pl = ffs.Planner(0)
flush = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
print(bench.run_c4(pl, 3, 3, flush, {}))
" > $D/ncu_c4.log 2>&1
timeout 900 python tools/shard_emulation.py > $D/shard.log 2>&1; cp gpurun_out/shard_emulation.json $D/ 2>/dev/null
timeout 600 python tools/seg_scaling.py > $D/seg_scaling.log 2>&1
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/issue_bench tools/issue_bench.cu && /tmp/issue_bench > $D/issue_bench.log 2>&1
