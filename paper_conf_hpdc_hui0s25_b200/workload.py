"""Seeded synthetic workloads for the pipeline-construction search.

This module only DRAWS inputs: profile tables, cluster free-slice state, request
batches, instance snapshots.  It holds none of the method's arithmetic (no stage
sums, no feasibility, no CV, no keys) and imports neither the CUDA binding nor the
oracle; both sides consume the arrays it returns.

Randomness is a counter-based SplitMix64 (seed ``0x5EED0000 + config_id``), vectorised
with numpy so that a 1M-request batch is drawn in well under a second.

Paper anchors for the recipe (P:<line> of /root/reference/PAPER.md):
  * MIG profiles 1g/2g/3g/4g/7g with 1/2/3/4/7 GPCs and 10/20/40/40/80 GB (Table 2,
    P:113-121); 1 "gb" = 1024 MiB (R14).
  * GPU partitions P1, P2, Hybrid (Table 7) plus whole-GPU 7g nodes.
  * Application chains of DNN components (Table 4): conv-class
    (super-resolution, segmentation, deblur, depth, U2-Net), transformer-class and
    heads.  Small/medium/large memory classes (Table 5).
  * SLO = 1.5 x the latency alone on the minimum MIG; requests carry the
    remaining budget (deadline minus waiting, P:364/P:374 -> DESIGN.md R9).
  * Inter-stage transfer of 1.7-44 ms per cut so that 2-3 stage pipelines land in the
    10-40 ms range of P:514.
  * Azure-Functions-shaped popularity: Zipf(1.0) over functions.
"""
from __future__ import annotations

from dataclasses import dataclass, field
import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
SEED_BASE = 0x5EED0000

# Table 2: order 1g, 2g, 3g, 4g, 7g
PROFILE_NAMES = ("1g.10gb", "2g.20gb", "3g.40gb", "4g.40gb", "7g.80gb")
PROFILE_GPCS = np.array([1, 2, 3, 4, 7], dtype=np.uint32)
PROFILE_CAP_MIB = np.array([10, 20, 40, 40, 80], dtype=np.uint32) * 1024
G1, G2, G3, G4, G7 = range(5)
GB = 1024  # MiB

# Table 7 GPU partitions, one list of profile ids per GPU
PART_P1 = [[G4, G2, G1]] * 8
PART_P2 = [[G3, G2, G2]] * 8
PART_HYBRID = [[G1] * 7] + [[G2, G2, G2, G1]] * 2 + [[G3, G4]] * 4 + [[G4, G2, G1]]
PART_7G = [[G7]] * 8
# 8-node block = 3xP1, 3xP2, 1xHybrid, 1x[7g]  (178 slices)
NODE_BLOCK = [PART_P1] * 3 + [PART_P2] * 3 + [PART_HYBRID] + [PART_7G]

# ABI record layouts (include/ffs.h); little-endian, natural alignment
SLICE_DTYPE = np.dtype([("node", "<u2"), ("gpu", "u1"), ("slice", "u1"), ("profile", "u1"),
                        ("busy", "u1"), ("pad", "<u2"), ("instance", "<i4")])
REQ_DTYPE = np.dtype([("func", "<u4"), ("node", "<u4")])
INST_DTYPE = np.dtype([("func", "<u4"), ("slice", "<i4"), ("flags", "u1"), ("pad", "u1", (3,)),
                       ("busy_us", "<u4"), ("last_used_us", "<u8")])
assert SLICE_DTYPE.itemsize == 12 and REQ_DTYPE.itemsize == 8 and INST_DTYPE.itemsize == 24

INST_PIPELINE = 1
INST_BUSY = 2


def _mix(z: np.ndarray) -> np.ndarray:
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


class SplitMix64:
    """Counter-based SplitMix64: draw i of a stream is mix(seed + (i+1)*golden)."""

    def __init__(self, seed: int):
        self.state = np.uint64(seed & 0xFFFFFFFFFFFFFFFF)
        self.count = 0

    def u64(self, n: int) -> np.ndarray:
        with np.errstate(over="ignore"):
            i = np.arange(self.count + 1, self.count + n + 1, dtype=np.uint64)
            out = _mix(self.state + i * GOLDEN)
        self.count += n
        return out

    def uniform(self, n: int, lo: float = 0.0, hi: float = 1.0) -> np.ndarray:
        u = (self.u64(n) >> np.uint64(11)).astype(np.float64) * (1.0 / (1 << 53))
        return lo + (hi - lo) * u

    def integers(self, lo: int, hi: int, n: int) -> np.ndarray:
        """Uniform integers in [lo, hi] inclusive."""
        span = np.uint64(hi - lo + 1)
        return (self.u64(n) % span).astype(np.int64) + lo

    def choice(self, probs: np.ndarray, n: int) -> np.ndarray:
        cdf = np.cumsum(probs) / np.sum(probs)
        return np.minimum(np.searchsorted(cdf, self.uniform(n), side="right"), len(probs) - 1)

    def sub(self, tag: int) -> "SplitMix64":
        return SplitMix64(int(_mix(np.array([int(self.state) ^ (tag * 0x2545F4914F6CDD1D & 0xFFFFFFFFFFFFFFFF)],
                                            dtype=np.uint64))[0]))


@dataclass
class Problem:
    """One planning input: profiles + profile table + cluster + requests."""
    name: str
    gpcs: np.ndarray
    cap_mib: np.ndarray
    comp_off: np.ndarray   # uint32 [F+1]
    lat_us: np.ndarray     # uint32 [C, P]
    mem_mib: np.ndarray    # uint32 [C]
    xfer_us: np.ndarray    # uint32 [C]  cost of a cut after component c (last one unused)
    load_us: np.ndarray    # uint32 [F]  warm -> MIG reload time
    n_nodes: int
    slices: np.ndarray     # SLICE_DTYPE [S] sorted by (node, gpu, slice)
    req: np.ndarray        # REQ_DTYPE [R]
    slo_us: np.ndarray     # uint32 [R] remaining latency budget B_r
    k_max: int = 4
    meta: dict = field(default_factory=dict)
    # throughput floor per function (R38, NEXT-2): every stage of a plan runs in at most
    # max_stage_us[f] us (= 10^6 / lambda_f); 0 = none; None = no floors at all
    max_stage_us: np.ndarray | None = None

    @property
    def P(self) -> int:
        return int(self.gpcs.shape[0])

    @property
    def F(self) -> int:
        return int(self.comp_off.shape[0] - 1)

    @property
    def R(self) -> int:
        return int(self.req.shape[0])

    def chain_len(self) -> np.ndarray:
        return np.diff(self.comp_off.astype(np.int64))

    def with_requests(self, req: np.ndarray, slo_us: np.ndarray) -> "Problem":
        d = dict(self.__dict__)
        d["req"] = np.ascontiguousarray(req, dtype=REQ_DTYPE)
        d["slo_us"] = np.ascontiguousarray(slo_us, dtype=np.uint32)
        return Problem(**d)

    def subset(self, idx: np.ndarray) -> "Problem":
        return self.with_requests(self.req[idx], self.slo_us[idx])


# ----------------------------------------------------------------------------------
# profile tables
# ----------------------------------------------------------------------------------
_FAMILY = {  # base latency on 7g (us), log-uniform, and the slow-down exponent alpha
    "conv": ((2000.0, 40000.0), (0.60, 0.95)),
    "transformer": ((1000.0, 8000.0), (0.40, 0.80)),
    "head": ((500.0, 3000.0), (0.10, 0.40)),
}


def _component_families(rng: SplitMix64, n: int) -> list[str]:
    kind = rng.choice(np.array([0.6, 0.25, 0.15]), 1)[0]
    if kind == 0:  # conv chain (SR / seg / deblur / depth / U2-Net), maybe with a head
        fam = ["conv"] * n
        if n >= 2 and rng.uniform(1)[0] < 0.5:
            fam[-1] = "head"
    elif kind == 1:  # BERT-class transformer layers
        fam = ["transformer"] * n
    else:
        pick = rng.choice(np.array([0.5, 0.35, 0.15]), n)
        fam = [("conv", "transformer", "head")[i] for i in pick]
    return fam


def _split_memory(rng: SplitMix64, total_mib: int, n: int, per_comp_max: int) -> np.ndarray:
    w = rng.uniform(n, 0.2, 1.0)
    m = np.maximum(1, np.floor(total_mib * w / w.sum())).astype(np.int64)
    for _ in range(64):  # push any excess above the per-component bound onto the others
        over = m > per_comp_max
        if not over.any():
            break
        excess = int((m[over] - per_comp_max).sum())
        m[over] = per_comp_max
        room = np.where(m < per_comp_max, per_comp_max - m, 0)
        if room.sum() == 0:
            break
        add = np.floor(excess * room / room.sum()).astype(np.int64)
        m += np.minimum(add, room)
    return m


def make_function(rng: SplitMix64, n: int, size_class: str, gpcs: np.ndarray = PROFILE_GPCS):
    """lat[c][p] = ceil(base7g_c * (7/g_p)^alpha_c) us; mem by Table 5 class."""
    fam = _component_families(rng, n)
    lat = np.zeros((n, gpcs.shape[0]), dtype=np.uint32)
    for c, f in enumerate(fam):
        (blo, bhi), (alo, ahi) = _FAMILY[f]
        base = float(np.exp(rng.uniform(1, np.log(blo), np.log(bhi))[0]))
        alpha = float(rng.uniform(1, alo, ahi)[0])
        lat[c] = np.ceil(base * (7.0 / gpcs.astype(np.float64)) ** alpha).astype(np.uint32)
    if size_class == "small":
        total, bound = int(rng.uniform(1, 1.0, 10.0)[0] * GB), 10 * GB
    elif size_class == "medium":
        total, bound = int(rng.uniform(1, 10.5, 20.0)[0] * GB), 10 * GB
    else:
        total, bound = int(rng.uniform(1, 21.0, 40.0)[0] * GB), 20 * GB
    mem = _split_memory(rng, total, n, bound).astype(np.uint32)
    out_mib = rng.uniform(n, 4.0, 256.0)
    xfer = (1000 + np.ceil(170.0 * out_mib)).astype(np.uint32)
    xfer[-1] = 0
    load = np.uint32(np.ceil(int(mem.sum()) * 40.0))  # ~25 GB/s host -> device reload
    return lat, mem, xfer, load


def _size_class(rng: SplitMix64, n: int, mix=(0.30, 0.35, 0.35)) -> str:
    c = ("small", "medium", "large")[rng.choice(np.array(mix), 1)[0]]
    if n == 1:
        return "small"
    if c == "large" and n < 2:
        return "medium"
    return c


def make_table(rng: SplitMix64, lengths, classes=None, mix=(0.30, 0.35, 0.35)):
    lats, mems, xfers, loads, cls = [], [], [], [], []
    for i, n in enumerate(lengths):
        c = classes[i] if classes is not None else _size_class(rng, int(n), mix)
        lat, mem, xfer, load = make_function(rng, int(n), c)
        lats.append(lat); mems.append(mem); xfers.append(xfer); loads.append(load); cls.append(c)
    comp_off = np.zeros(len(lengths) + 1, dtype=np.uint32)
    comp_off[1:] = np.cumsum(np.asarray(lengths, dtype=np.int64))
    return (comp_off, np.concatenate(lats).astype(np.uint32), np.concatenate(mems).astype(np.uint32),
            np.concatenate(xfers).astype(np.uint32), np.asarray(loads, dtype=np.uint32), cls)


# ----------------------------------------------------------------------------------
# cluster state
# ----------------------------------------------------------------------------------
# Busy probability of a slice relative to the node's load rho, by profile: under
# monolithic placement the large slices are the ones kept occupied while 1g/2g
# slices idle (Fig. 3(b), "only the 4g.40gb MIG slices are actively utilized").
BUSY_WEIGHT = np.array([0.3, 0.9, 2.0, 2.0, 2.0])


def make_slices(rng: SplitMix64, node_parts, rho=None, rho_range=(0.3, 0.9)) -> np.ndarray:
    rows = []
    for v, part in enumerate(node_parts):
        r = rho if rho is not None else float(rng.uniform(1, *rho_range)[0])
        for g, gpu in enumerate(part):
            pb = np.minimum(0.98, r * BUSY_WEIGHT[np.asarray(gpu)])
            busy = rng.uniform(len(gpu)) < pb
            for s, p in enumerate(gpu):
                rows.append((v, g, s, p, int(busy[s]), 0, -1))
    return np.array(rows, dtype=SLICE_DTYPE)


# ----------------------------------------------------------------------------------
# requests
# ----------------------------------------------------------------------------------
def slo_per_function(comp_off, lat, mem, cap=PROFILE_CAP_MIB, scale=1.5, basis="component"):
    """SLO_f = floor(scale * t_f), t_f = latency "alone ... on the minimum MIG
    instances, as shown in Table 5".  basis="component" (default, R9) reads the
    minimum MIG as Table 5's FluidFaaS column: the smallest profile that holds every
    component, t_f = sum of component latencies on it.  basis="monolithic" reads it as
    the Baseline column: the smallest profile holding the whole function.  7g if none.
    Returns (slo, t_f, t_fastest) with t_fastest the fastest 1-stage latency."""
    F = comp_off.shape[0] - 1
    slo = np.zeros(F, dtype=np.int64)
    t_f = np.zeros(F, dtype=np.int64)
    t_fast = np.zeros(F, dtype=np.int64)
    order = np.lexsort((np.arange(cap.shape[0]), cap))  # by capacity, then id
    for f in range(F):
        a, b = int(comp_off[f]), int(comp_off[f + 1])
        m = mem[a:b].astype(np.int64)
        need = int(m.max()) if basis == "component" else int(m.sum())
        pmin = next((int(p) for p in order if need <= int(cap[p])), int(order[-1]))
        t_f[f] = int(lat[a:b, pmin].astype(np.int64).sum())
        t_fast[f] = int(lat[a:b].astype(np.int64).sum(axis=0).min())
        slo[f] = int(np.floor(scale * t_f[f]))
    return slo, t_f, t_fast


def make_requests(rng: SplitMix64, R: int, F: int, n_nodes: int, slo_f, t_f, t_fast,
                  zipf_s=1.0, p_infeasible=0.01, p_loose=0.05):
    rank = np.arange(1, F + 1, dtype=np.float64)
    pop = rank ** (-zipf_s)
    perm = np.argsort(rng.u64(F))  # popularity independent of chain length
    func = perm[rng.choice(pop, R)].astype(np.uint32)
    node = rng.integers(0, n_nodes - 1, R).astype(np.uint32)
    slo = slo_f[func].astype(np.float64)
    wait = rng.uniform(R, 0.0, 0.5) * slo
    u = rng.uniform(R)
    loose = (u >= p_infeasible) & (u < p_infeasible + p_loose)
    budget = np.where(loose, np.floor(3.0 * t_f[func]) - wait, slo - wait)
    forced = u < p_infeasible  # below the fastest possible 1-stage latency
    budget = np.where(forced, np.floor(rng.uniform(R, 0.3, 0.95) * t_fast[func]), budget)
    budget = np.clip(np.floor(budget), 0, 0xFFFFFFFF).astype(np.uint32)
    req = np.zeros(R, dtype=REQ_DTYPE)
    req["func"] = func
    req["node"] = node
    return req, budget


# ----------------------------------------------------------------------------------
# the five configs (BASELINE.json "configs")
# ----------------------------------------------------------------------------------
def _problem(name, rng, lengths, node_parts, R, rho=None, k_max=4, classes=None, mix=(0.30, 0.35, 0.35),
             rho_range=(0.3, 0.9)):
    comp_off, lat, mem, xfer, load, cls = make_table(rng.sub(1), lengths, classes, mix)
    slices = make_slices(rng.sub(2), node_parts, rho, rho_range)
    slo_f, t_f, t_fast = slo_per_function(comp_off, lat, mem)
    req, slo = make_requests(rng.sub(3), R, len(lengths), len(node_parts), slo_f, t_f, t_fast)
    return Problem(name=name, gpcs=PROFILE_GPCS.copy(), cap_mib=PROFILE_CAP_MIB.copy(), comp_off=comp_off,
                   lat_us=lat, mem_mib=mem, xfer_us=xfer, load_us=load, n_nodes=len(node_parts),
                   slices=slices, req=req, slo_us=slo, k_max=k_max,
                   meta={"classes": cls, "slo_f": slo_f, "t_f": t_f, "t_fast": t_fast})


def config1(seed: int | None = None) -> Problem:
    """C1: 1 function, 4-component medium chain (sum ~18 GB, each <= 10 GB), one GPU
    of 7 x 1g.10gb (Table 2 max count, Hybrid row P:520), all free, 16 requests with
    budgets spread from infeasible to 3 x SLO."""
    rng = SplitMix64(SEED_BASE + 1 if seed is None else seed)
    lat, mem, xfer, load = make_function(rng.sub(1), 4, "medium")
    comp_off = np.array([0, 4], dtype=np.uint32)
    slices = make_slices(rng.sub(2), [[[G1] * 7]], rho=0.0)
    slo_f, t_f, t_fast = slo_per_function(comp_off, lat, mem)
    lo, hi = 0.5 * float(t_fast[0]), 3.0 * float(slo_f[0])
    budgets = np.floor(lo + (hi - lo) * np.arange(16) / 15.0).astype(np.uint32)
    req = np.zeros(16, dtype=REQ_DTYPE)
    return Problem(name="C1", gpcs=PROFILE_GPCS.copy(), cap_mib=PROFILE_CAP_MIB.copy(), comp_off=comp_off,
                   lat_us=lat, mem_mib=mem, xfer_us=xfer, load_us=np.array([load], dtype=np.uint32), n_nodes=1,
                   slices=slices, req=req, slo_us=budgets, k_max=4,
                   meta={"classes": ["medium"], "slo_f": slo_f, "t_f": t_f, "t_fast": t_fast})


def config1b(seed: int | None = None) -> Problem:
    """C1b: the C1 function on one GPU of each Table 7 pattern with random occupancy."""
    base = config1(seed)
    rng = SplitMix64((SEED_BASE + 11) if seed is None else seed + 11)
    gpus = [[G4, G2, G1], [G3, G2, G2], [G1] * 7, [G2, G2, G2, G1], [G3, G4], [G7]]
    slices = make_slices(rng, [[g] for g in gpus], rho=0.4)
    R = 16 * len(gpus)
    req = np.zeros(R, dtype=REQ_DTYPE)
    req["node"] = np.repeat(np.arange(len(gpus)), 16)
    slo = np.tile(base.slo_us, len(gpus))
    p = base.with_requests(req, slo)
    p.slices, p.n_nodes, p.name = slices, len(gpus), "C1b"
    return p


def config2(seed: int | None = None, R: int = 4096) -> Problem:
    """C2: 6 functions n in {3,3,5,6,8,12} (App0/App1 3-chains, App3 linearised 5,
    ResNet-50 6, VGG-16 8, BERT-base 12), one node of 8 Hybrid GPUs (26 slices),
    rho = 0.5, 4096 requests."""
    rng = SplitMix64(SEED_BASE + 2 if seed is None else seed)
    classes = ["medium", "large", "medium", "small", "medium", "large"]  # Table 5 variants
    return _problem("C2", rng, [3, 3, 5, 6, 8, 12], [PART_HYBRID], R, rho=0.5, classes=classes)


def config3(seed: int | None = None, R: int = 65536) -> Problem:
    """C3: 20 functions n in U[3,24], 8 nodes = 64 GPUs (3xP1, 3xP2, Hybrid, 7g)."""
    rng = SplitMix64(SEED_BASE + 3 if seed is None else seed)
    lengths = rng.sub(9).integers(3, 24, 20)
    return _problem("C3", rng, lengths, NODE_BLOCK, R)


def config5(seed: int | None = None, R: int = 1 << 20) -> Problem:
    """C5: 64 functions n in U[3,32], 128 nodes = 1024 GPUs, 1M requests."""
    rng = SplitMix64(SEED_BASE + 5 if seed is None else seed)
    lengths = rng.sub(9).integers(3, 32, 64)
    return _problem("C5", rng, lengths, NODE_BLOCK * 16, R)


# ----------------------------------------------------------------------------------
# C4: hotness-aware eviction snapshots
# ----------------------------------------------------------------------------------
@dataclass
class EvictWorkload:
    problem: Problem            # profile table + cluster (32 nodes) + per-tick loads
    inst: np.ndarray            # INST_DTYPE, all ticks concatenated
    tick_off: np.ndarray        # uint32 [T+1]
    now_us: np.ndarray          # uint64 [T]
    req_tick: np.ndarray        # uint32 [R] tick of each load request (sorted)
    window_us: int = 10_000_000
    util_thr_pct: int = 30
    cold_after_us: int = 600_000_000


def config4(seed: int | None = None, T: int = 4096, n_funcs: int = 200) -> EvictWorkload:
    """C4: 32 nodes = 256 GPUs (4 x the C3 block, 712 slices), 200 warm functions each
    with at most one time-sharing instance plus 0-4 exclusive-hot instances,
    T tick snapshots 100 ms apart (window 10 s), and 1-50 loads per tick."""
    rng = SplitMix64(SEED_BASE + 4 if seed is None else seed)
    lengths = rng.sub(9).integers(3, 12, n_funcs)
    base = _problem("C4", rng, lengths, NODE_BLOCK * 4, 1, rho_range=(0.5, 0.95))
    S = base.slices.shape[0]
    r = rng.sub(5)
    window = 10_000_000
    t0 = 3_600_000_000
    now = (t0 + 100_000 * np.arange(T, dtype=np.uint64)).astype(np.uint64)
    # per function: hotness (Zipf popularity) and number of exclusive-hot instances
    hot_n = r.integers(0, 4, n_funcs)
    util_mean = r.uniform(n_funcs, 0.02, 0.6)
    per_tick = n_funcs + int(hot_n.sum())
    n = per_tick * T
    func = np.concatenate([np.arange(n_funcs), np.repeat(np.arange(n_funcs), hot_n)]).astype(np.uint32)
    func = np.tile(func, T)
    is_ts = np.tile(np.concatenate([np.ones(n_funcs, bool), np.zeros(int(hot_n.sum()), bool)]), T)
    tick = np.repeat(np.arange(T), per_tick)
    inst = np.zeros(n, dtype=INST_DTYPE)
    inst["func"] = func
    resident = r.uniform(n) < np.where(is_ts, 0.6, 0.97)
    inst["slice"] = np.where(resident, r.integers(0, S - 1, n), -1).astype(np.int32)
    flags = np.where(~is_ts & (r.uniform(n) < 0.3), INST_PIPELINE, 0)
    flags |= np.where(r.uniform(n) < 0.15, INST_BUSY, 0)
    inst["flags"] = flags.astype(np.uint8)
    util = np.clip(util_mean[func] * r.uniform(n, 0.3, 2.0), 0.0, 1.0)
    inst["busy_us"] = np.floor(util * window).astype(np.uint32)
    idle = np.floor(r.uniform(n) ** 3 * 900_000_000).astype(np.uint64)  # some beyond 10 min
    inst["last_used_us"] = now[tick] - idle
    tick_off = (np.arange(T + 1) * per_tick).astype(np.uint32)
    # loads (requests) per tick, 1..50, each on a random node
    loads = r.integers(1, 50, T)
    R = int(loads.sum())
    req_tick = np.repeat(np.arange(T), loads).astype(np.uint32)
    slo_f, t_f, t_fast = base.meta["slo_f"], base.meta["t_f"], base.meta["t_fast"]
    req, slo = make_requests(r.sub(7), R, n_funcs, base.n_nodes, slo_f, t_f, t_fast)
    prob = base.with_requests(req, slo)
    prob.name = "C4"
    return EvictWorkload(problem=prob, inst=inst, tick_off=tick_off, now_us=now, req_tick=req_tick,
                         window_us=window)


CONFIGS = {1: config1, 2: config2, 3: config3, 5: config5}


# ----------------------------------------------------------------------------------
# NEXT-4: request trace for the time-sharing simulator
# ----------------------------------------------------------------------------------
@dataclass
class SimTrace:
    problem: Problem           # profile table + cluster (busy slices are other tenants)
    req_off: np.ndarray        # uint32 [n_nodes * T + 1] CSR: requests of (node, tick)
    req_func: np.ndarray       # uint32 [n_req]
    req_budget: np.ndarray     # uint32 [n_req] latency budget (SLO) of the request
    T: int
    tick_us: int = 100_000
    window_ticks: int = 100    # 10 s utilisation window
    t0_us: int = 1_000_000_000


def sim_trace(seed: int | None = None, T: int = 4096, n_funcs: int = 200, nodes=None,
              rate_scale: float = 1.0) -> SimTrace:
    """Azure-shaped arrivals: Zipf(1) function popularity, per (node,
    function) bursty on/off Poisson rates; budgets = SLO_f."""
    rng = SplitMix64(SEED_BASE + 6 if seed is None else seed)
    node_parts = NODE_BLOCK * 4 if nodes is None else nodes
    lengths = rng.sub(9).integers(3, 12, n_funcs)
    base = _problem("SIM", rng, lengths, node_parts, 1, rho_range=(0.2, 0.6))
    N = base.n_nodes
    r = rng.sub(7)
    pop = (np.arange(1, n_funcs + 1, dtype=np.float64) ** -1.0)
    pop = pop[np.argsort(r.u64(n_funcs))]
    lam = 0.05 * rate_scale * pop / pop.max()                       # requests per tick per node
    on = r.uniform(N * n_funcs).reshape(N, n_funcs) < 0.5
    # bursty: a function alternates on/off phases of 30..300 ticks per node
    phase = r.integers(30, 300, N * n_funcs).reshape(N, n_funcs)
    counts = np.zeros((N, T), dtype=np.int64)
    funcs_per = [[None] * T for _ in range(N)]
    u = r.uniform(N * T * n_funcs).reshape(N, T, n_funcs)
    for t in range(T):
        flip = (t % phase) == 0
        on = np.where(flip & (t > 0), ~on, on)
        p = np.where(on, lam[None, :] * 3.0, lam[None, :] * 0.2)      # on: 3x, off: 0.2x
        hit = u[:, t, :] < p
        for v in range(N):
            fs = np.nonzero(hit[v])[0]
            funcs_per[v][t] = fs
            counts[v, t] = fs.shape[0]
    req_off = np.zeros(N * T + 1, dtype=np.uint32)
    req_off[1:] = np.cumsum(counts.reshape(-1))
    req_func = np.concatenate([funcs_per[v][t] for v in range(N) for t in range(T)]).astype(np.uint32) \
        if req_off[-1] else np.zeros(0, np.uint32)
    slo_f = base.meta["slo_f"]
    req_budget = slo_f[req_func].astype(np.uint32)
    return SimTrace(problem=base, req_off=req_off, req_func=req_func, req_budget=req_budget, T=T)


def with_throughput_floor(prob: Problem, seed: int = 0x5EEDF100, lo: float = 0.35, hi: float = 1.0,
                          none_frac: float = 0.25) -> Problem:
    """A copy of `prob` whose functions carry a throughput floor (R38, NEXT-2): instances
    sized for the function's load lambda_f ("an instance requiring 4g.40gb"), i.e.
    max_stage_us[f] = floor(u_f * t_f) with t_f the 1-stage latency on the SLO basis profile
    and u_f ~ U[lo, hi] -- below 1, only a faster slice or a pipeline (whose bottleneck is a
    fraction of the chain) serves f.  A fraction `none_frac` of the functions has no floor."""
    rng = SplitMix64(seed)
    F = prob.F
    t_f = np.asarray(prob.meta["t_f"], dtype=np.float64)
    u = rng.uniform(F, lo, hi)
    fl = np.floor(u * t_f).astype(np.uint32)
    fl[rng.sub(1).uniform(F) < none_frac] = 0
    d = dict(prob.__dict__)
    d["max_stage_us"] = np.maximum(fl, 0).astype(np.uint32)
    d["name"] = prob.name + "+floor"
    return Problem(**d)


# ----------------------------------------------------------------------------------
# NEXT-1 DAG functions (R40-R43): series of units, a unit is one component or
# a fork/join block of parallel branches (expanded image classification "is
# extended with two branches to form a DAG")
# ----------------------------------------------------------------------------------
class Cond(list):
    """A conditional unit in a DAG shape (R48, App 3): alternative branches, exactly
    one runs per request; a branch of length 0 is "pass"."""


@dataclass
class DagTable:
    """Unit structure of every function of a Problem (include/ffs.h ffs_dag_table)."""
    unit_off: np.ndarray   # uint32 [F+1]
    unit_nb: np.ndarray    # uint8  [U] branches 1..4 (1 = one component)
    unit_bend: np.ndarray  # uint8  [U, 4] function-relative exclusive end of branch j (0 unused)
    unit_cond: np.ndarray | None = None  # uint8 [U] 1 = conditional unit (R48), None = none


    def units(self, f: int) -> list[list[tuple[int, int]]]:
        """Function f's units as lists of (first, end) component ranges per branch."""
        out, c = [], 0
        for u in range(int(self.unit_off[f]), int(self.unit_off[f + 1])):
            br = []
            for j in range(int(self.unit_nb[u])):
                e = int(self.unit_bend[u, j])
                br.append((c, e))
                c = e
            out.append(br)
        return out


def chain_dag(prob: Problem) -> DagTable:
    """The DAG of a plain chain: every component is its own unit."""
    n = prob.chain_len()
    unit_off = np.zeros(prob.F + 1, dtype=np.uint32)
    unit_off[1:] = np.cumsum(n)
    bend = np.zeros((int(unit_off[-1]), 4), dtype=np.uint8)
    bend[:, 0] = np.concatenate([np.arange(1, int(x) + 1) for x in n])
    return DagTable(unit_off, np.ones(int(unit_off[-1]), dtype=np.uint8), bend)


def make_dag_shapes(rng: SplitMix64, F: int, units=(3, 8), p_block=0.35, branches=(2, 2), br_len=(1, 3),
                    p_cond: float = 0.0):
    """Per function: a list of units, each a list of branch lengths; with probability
    p_cond a unit is conditional (App 3's "if low resolution: super resolution; else:
    pass"): a Cond of one 1..2-component branch and a pass."""
    shapes = []
    c_rng = rng.sub(17)  # separate stream: p_cond = 0 reproduces the round-1 shapes
    for _ in range(F):
        m = int(rng.integers(units[0], units[1], 1)[0])
        u_list = []
        for _ in range(m):
            if float(rng.uniform(1)[0]) < p_block:
                nb = int(rng.integers(branches[0], branches[1], 1)[0])
                u_list.append([int(x) for x in rng.integers(br_len[0], br_len[1], nb)])
            else:
                u_list.append([1])
            if p_cond and float(c_rng.uniform(1)[0]) < p_cond and len(u_list[-1]) == 1:
                u_list[-1] = Cond([int(c_rng.integers(1, 2, 1)[0]), 0])
        shapes.append(u_list)
    return shapes


def dag_table(shapes) -> DagTable:
    """Shapes: per function a list of units, each a list of branch lengths (a fork/join
    block when > 1) or a Cond of alternative branch lengths (0 = pass)."""
    unit_off = np.zeros(len(shapes) + 1, dtype=np.uint32)
    unit_off[1:] = np.cumsum([len(s) for s in shapes])
    U = int(unit_off[-1])
    nb = np.zeros(U, dtype=np.uint8)
    bend = np.zeros((U, 4), dtype=np.uint8)
    cond = np.zeros(U, dtype=np.uint8)
    u = 0
    for s in shapes:
        c = 0
        for br in s:
            nb[u] = len(br)
            cond[u] = isinstance(br, Cond)
            for j, L in enumerate(br):
                c += L
                bend[u, j] = c
            u += 1
    return DagTable(unit_off, nb, bend, cond if cond.any() else None)


def dag_config(seed: int | None = None, R: int = 1 << 16, F: int = 32, node_parts=None, k_max: int = 4,
               p_block: float = 0.35, units=(3, 8), branches=(2, 2), p_cond: float = 0.0) -> tuple[Problem, DagTable]:
    """CD: DAG functions (3..8 units, a unit a 2-branch block with probability 0.35,
    branches of 1..3 components) on the C3 cluster (8 nodes = 64 GPUs), Azure-shaped
    requests as C3.  Components and budgets follow the chain recipe (make_function,
    R9 SLO on the summed single-slice latency)."""
    rng = SplitMix64(SEED_BASE + 6 if seed is None else seed)
    shapes = make_dag_shapes(rng.sub(8), F, units, p_block, branches, p_cond=p_cond)
    lengths = [sum(sum(br) for br in s) for s in shapes]
    prob = _problem("CD", rng, lengths, NODE_BLOCK if node_parts is None else node_parts, R, k_max=k_max)
    return prob, dag_table(shapes)
