set -x
mkdir -p gpurun_out/r2i
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2i/build.log 2>&1
timeout 600 python tools/seg_scaling.py > gpurun_out/r2i/seg_scaling.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_evict_ticks" --launch-skip 5 --launch-count 1 -f -o gpurun_out/r2i/prof_c4 python -c "
import sys; sys.path.insert(0,'.')
import bench, torch
from paper_conf_hpdc_hui0s25_b200 import ffs
pl = ffs.Planner(0)
flush = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
print(bench.run_c4(pl, 3, 3, flush, {}))
" > gpurun_out/r2i/ncu_c4.log 2>&1
