"""Launched by tests/test_gpu_dist.py under torchrun: the sharded step (dist.plan_step)
on the real CUDA kernels with WORLD_SIZE ranks sharing the available GPU(s); rank 0
checks the combined keys and the gathered plan slices against a single-rank run."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

from paper_conf_hpdc_hui0s25_b200 import ffs, dist as D, workload as W  # noqa: E402

backend = os.environ.get("FFS_DIST_BACKEND", "gloo")
rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
dev = int(os.environ.get("LOCAL_RANK", "0")) % torch.cuda.device_count()
torch.cuda.set_device(dev)
dist.init_process_group(backend)
prob = W.config3(R=8192)
pl = ffs.Planner(dev)
pl.stage(prob)
req, slo = ffs.to_device(prob)
lo, hi = D.request_slice(prob.R, rank, world)
ref_keys = pl.plan_keys(req, slo, prob.k_max)          # single rank, whole task space
ref_plans = pl.plan_decode(req, slo, ref_keys, prob.k_max).cpu().numpy()
ref_keys = ref_keys.cpu().numpy()
for shard in ("requests", "candidates"):
    keys = torch.full((prob.R,), np.iinfo(np.int64).max, dtype=torch.int64, device="cuda")
    plans = torch.empty((hi - lo, 80), dtype=torch.uint8, device="cuda")
    D.plan_step(pl, req, slo, prob.k_max, rank, world, keys, plans, shard=shard)
    torch.cuda.synchronize()
    mine = (lo, hi, plans.cpu().numpy().tobytes(), keys.cpu().numpy().tobytes())
    got = [None] * world
    dist.all_gather_object(got, mine)
    if rank == 0:
        for lo_, hi_, pb, kb in got:
            k = np.frombuffer(kb, np.int64)
            if shard == "candidates":  # every rank holds the combined keys of the batch
                assert np.array_equal(k, ref_keys)
            else:                      # a rank holds the keys of its own requests
                assert np.array_equal(k[lo_:hi_], ref_keys[lo_:hi_])
            assert np.array_equal(np.frombuffer(pb, np.uint8).reshape(-1, 80), ref_plans[lo_:hi_])
        assert got[0][0] == 0 and got[-1][1] == prob.R
        print(f"dist-run ok world={world} backend={backend} shard={shard}")
dist.destroy_process_group()
