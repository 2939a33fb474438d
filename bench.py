#!/usr/bin/env python
"""Benchmark of the B200 Boids step (one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload c4] [--impl ours|reference]
    torchrun --nproc-per-node N --master-addr 127.0.0.1 bench.py --gpus N ...

A "step" is one synchronous Boids update of ALL agents (every SURVEY.md 8(a)
row: [a1 all-gather at N>1] -> a3 search -> a4 split merge -> a5 steering ->
a6 modification; a2 binning in grid mode), through the C ABI of libboids.so.

* value      agent-steps/s of the whole job = n * K / max-over-ranks device time,
             CUDA events on the launching stream, L2 flushed (256 MiB write)
             before every timed step (the state of every config fits in L2).
* e2e        the same metric through the public C ABI with HOST buffers: every
             step boids_set_state (H2D) + step + boids_get_state (D2H), wall clock.
* roofline   the search kernel of the path the library reports it ran
             (boids_info.last_path: k_sym -- its prologue k_sym_prep reported apart
             and combined --, k_bound + k_scan, k_grid, k_small):
             algorithmic FP32 lane-ops per launch (8 per evaluated pair,
             DESIGN.md sec 5) / its mean launch duration (library-side CUDA
             events on the handle's stream; inside the timed region, or with
             --kernel-timing pass in a profiled pass of K steps right after it),
             against the FP32 SIMT peak 148 SMs x 128 lanes x sm_max_mhz.
* update_roofline / update_standalone / binning_roofline  the update and
             binning kernels against the measured HBM copy bandwidth.
* cpu_baseline  the CPU oracle (oracle/, single thread) on a bounded sample of
             the same workload: full O(n) search + steer + modify for each sampled
             agent, extrapolated per agent-step (rank 0, N=1 only).
* --impl reference  times that oracle alone (the tier's reference arm).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import workloads as W  # noqa: E402

METRIC = json.load(open(os.path.join(ROOT, "BASELINE.json")))["metric"]
UNIT = "agent-steps/s"
LANES_PER_SM = 128
OPS_PER_PAIR = 8  # 3 sub + 3 mul + 2 add, no FMA


def peaks():
    p = {}
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        p = json.load(open(path))
    return p


def env_rank():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


class ClockSampler:
    """Samples SM clock + throttle reasons via NVML while the timed region runs."""

    def __init__(self, dev_index: int, period: float = 0.005):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self.period = period
        self._stop = threading.Event()
        self._t = None
        try:
            import pynvml

            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(dev_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    _REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
        0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
        0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting",
    }

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self._REASONS.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.nv:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *exc):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": float(np.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def cpu_oracle_rate(cfg: W.Config, agents: int, seed: int = 1):
    """Oracle (single thread) on `agents` sampled agents of the config's initial state."""
    import oracle

    p = oracle.default_params(init_mode=cfg.init_mode, search_mode=cfg.search_mode)
    s = oracle.init(cfg.n, p, seed=seed)
    ag = W.sample_agents(cfg.n, agents, seed=seed)
    t = time.perf_counter()
    oracle.step_sample(s, ag, float(W.DT), p)
    dt = time.perf_counter() - t
    return len(ag) / dt, len(ag), dt


def cpu_oracle_rate_threads(cfg: W.Config, agents_per_thread: int, threads: int, seed: int = 1):
    """The same oracle over all host cores: the seeded sample split across
    `threads` Python threads, each calling the C oracle (ctypes releases the GIL)
    on its own slice of agents (the per-agent functions
    partitioned over the cores, no GPU involved)."""
    import threading

    import oracle

    p = oracle.default_params(init_mode=cfg.init_mode, search_mode=cfg.search_mode)
    s = oracle.init(cfg.n, p, seed=seed)
    ag = W.sample_agents(cfg.n, min(cfg.n, agents_per_thread * threads), seed=seed)
    parts = np.array_split(ag, threads)
    ts = [threading.Thread(target=oracle.step_sample, args=(s, part, float(W.DT), p)) for part in parts]
    t = time.perf_counter()
    for th in ts:
        th.start()
    for th in ts:
        th.join()
    dt = time.perf_counter() - t
    return len(ag) / dt, len(ag), dt


def cpu_sample_size(cfg: W.Config, seconds: float) -> int:
    """Agents per sample for ~`seconds` of oracle work (about 1 ns per candidate pair,
    measured on the GPU box: profiles/r1j bench lines)."""
    return int(max(64, min(cfg.n, seconds / (1e-9 * cfg.n))))


def run_reference(args, cfg):
    rank, world, _ = env_rank()
    if rank != 0:
        return 0
    m = cpu_sample_size(cfg, 1.0)
    for _ in range(args.warmup):
        cpu_oracle_rate(cfg, max(64, m // 8))
    times, agents = [], 0
    for k in range(args.steps):
        _, agents, dt = cpu_oracle_rate(cfg, m, seed=1)
        times.append(dt)
    total = float(np.sum(times))
    value = agents * args.steps / total
    sample = (f"{agents} of {cfg.n} agents per step (seeded sample), each a full O(n) search + steer + "
              f"modify from the config's initial state; {args.steps} steps")
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": total / args.steps * 1e3,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic", "config": dict(config_dict(cfg, args.gpus), think_every=max(1, args.think)),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    emit(line)
    return 0


def config_dict(cfg: W.Config, gpus: int):
    return {"workload": cfg.name, "desc": cfg.desc, "n": cfg.n,
            "search": "grid" if cfg.search_mode else "brute",
            "init": "world_ball_r50" if cfg.init_mode else "opensteer_ball_r20",
            "parallelism": f"agents sharded by index over {gpus} GPU(s), NCCL all-gather of pos+fwd per step"
            if gpus > 1 else "single GPU",
            "dt": float(W.DT), "seed": 1, "l2": "flushed (256 MiB write) before every timed step"}


_OUT = None


def emit(line: dict):
    """Print the one JSON line on the real stdout (fd 1 is redirected to stderr
    during the run so library banners, e.g. NCCL's version line, cannot mix in)."""
    os.write(_OUT, (json.dumps(line) + "\n").encode())


def main():
    global _OUT
    sys.stdout.flush()
    _OUT = os.dup(1)
    os.dup2(2, 1)
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="c4", choices=sorted(W.CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--cpu-seconds", type=float, default=10.0, help="oracle sample size (seconds of CPU work)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true", help="skip the e2e leg (profiling runs)")
    ap.add_argument("--kernel", type=int, default=0, help="0 fused (default), 1 two-kernel simple path")
    ap.add_argument("--think", type=int, default=1,
                    help="think frequency k (skipThink, P:424): each agent searches every k-th step")
    ap.add_argument("--no-sym", action="store_true",
                    help="single-GPU brute force: evaluate every ordered pair (k_scan) instead of each "
                         "unordered pair once (k_sym, default)")
    ap.add_argument("--kernel-timing", default="live", choices=["live", "pass"],
                    help="live (default): CUDA events bracket the search kernel inside the timed region; "
                         "pass: the timed region runs uninstrumented and the search kernel is timed with "
                         "events in a profiled pass of K steps right after (events inside a CUDA graph break "
                         "its PDL edges: at n <= 16384 that perturbs the step time itself)")
    ap.add_argument("--graph", type=int, default=0,
                    help="1: warm steps replay captured CUDA graphs (BOIDS_OPT_GRAPH); 0 (default): eager launches "
                         "(measured faster per flushed step on B200, DESIGN.md sec 5)")
    ap.add_argument("--force-shard", action="store_true",
                    help="use the multi-GPU code path (NCCL process group + sharded handles) even at N=1")
    args = ap.parse_args()
    cfg = W.CONFIGS[args.workload]
    if args.warmup < 3:
        args.warmup = 3  # timing rule: at least 3 warm-up steps
    if args.think > 1 and args.warmup < args.think + 1:
        args.warmup = args.think + 1  # steady state: every agent has thought once
    if args.impl == "reference":
        return run_reference(args, cfg)

    import torch

    rank, world, local = env_rank()
    if world != args.gpus:
        args.gpus = world
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist = None
    if world > 1 or args.force_shard:
        import torch.distributed as dist

        if "MASTER_ADDR" not in os.environ:
            os.environ["MASTER_ADDR"], os.environ["MASTER_PORT"] = "127.0.0.1", "29533"
        dist.init_process_group("nccl", rank=rank, world_size=world, device_id=dev)

    import paper_conf_ipps_breitbart09_b200 as pk
    from paper_conf_ipps_breitbart09_b200 import abi
    from paper_conf_ipps_breitbart09_b200.shard import ShardedFlock

    params = pk.boids_default_params(init_mode=cfg.init_mode, search_mode=cfg.search_mode,
                                     think_every=max(1, args.think))
    dt = float(W.DT)
    if dist is not None:
        # brute force: sym-shards (the unordered-pair triangle split over the ranks) unless --no-sym
        fl = ShardedFlock(cfg.n, params, seed=1, kernel=args.kernel, sym=not args.no_sym)
        h = fl.h
        step = lambda: fl.step(dt, 1)  # noqa: E731
        nloc = fl.hi - fl.lo
    else:
        fl = pk.Flock(cfg.n, params, seed=1, kernel=args.kernel, symmetric=not args.no_sym)
        h = fl.h
        abi.boids_set_option(h, abi.BOIDS_OPT_GRAPH, args.graph)
        step = lambda: fl.step(dt, 1)  # noqa: E731
        nloc = cfg.n

    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream()

    def barrier():
        if dist is not None:
            dist.barrier()

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()

    # ---------------- timed region: K steps, L2 flushed before each ----------------
    live = args.kernel_timing == "live"
    # events around the search launches only (level 2), or none (kernel timing in a later pass)
    abi.boids_set_option(h, abi.BOIDS_OPT_PROFILE, 2 if live else 0)
    abi.boids_get_profile(h, reset=True)
    info0 = abi.boids_info(h)
    launches0 = info0.launches
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        for k in range(args.steps):
            flush.fill_(float(k))
            ev[k][0].record(stream)
            step()
            ev[k][1].record(stream)
        torch.cuda.synchronize()
        barrier()
    info1 = abi.boids_info(h)
    launches = info1.launches - launches0
    prof = abi.boids_get_profile(h, reset=True)
    abi.boids_set_option(h, abi.BOIDS_OPT_PROFILE, 0)
    ms = float(sum(a.elapsed_time(b) for a, b in ev))
    grid_pairs = info1.grid_pairs - info0.grid_pairs  # grid search work of the steps `prof` timed
    path = int(info1.last_path)
    if not live:  # the search kernel timed in a profiled pass of K steps right after the timed region
        abi.boids_set_option(h, abi.BOIDS_OPT_PROFILE, 2)
        abi.boids_get_profile(h, reset=True)
        ip0 = abi.boids_info(h)
        for k in range(args.steps):
            flush.fill_(float(k))
            step()
        torch.cuda.synchronize()
        prof = abi.boids_get_profile(h, reset=True)
        abi.boids_set_option(h, abi.BOIDS_OPT_PROFILE, 0)
        ip1 = abi.boids_info(h)
        grid_pairs, path = ip1.grid_pairs - ip0.grid_pairs, int(ip1.last_path)
    if dist is not None:
        t = torch.tensor([ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    value = cfg.n * args.steps / (ms / 1e3)

    # ---------------- roofline of the dominant kernel ----------------
    grid = cfg.search_mode == 1
    kname = "grid_search" if grid else "fused_or_search"
    k_ms, k_n = prof[kname]
    k_ms_per = k_ms / max(k_n, 1)
    think = max(1, args.think)
    # the library reports which search path the timed steps ran (boids_info.last_path)
    sym = path == abi.BOIDS_PATH_SYM
    if grid:  # algorithmic work of the grid search: pairs over the 27-cell stencils (device counter)
        pairs_per_launch = float(grid_pairs) / max(k_n, 1)
        pairs_note = " (27-cell stencil candidates, device counter)"
    elif sym:  # k_sym: every unordered pair once, tested against both agents' limits
        pairs_per_launch = float(cfg.n) * float(cfg.n - 1) / 2 / world
        pairs_note = " (n(n-1)/2 unordered pairs: d2 is symmetric, each evaluated once for both agents)"
        if world > 1:
            pairs_note += f"; this rank's 1/{world} share of the triangle (sym-shards)"
    else:  # every thinking agent against all n (think mode: 1/k of the agents per step)
        pairs_per_launch = float(nloc) * float(cfg.n) / think
        pairs_note = " (n_local x n ordered pairs)"
    achieved = OPS_PER_PAIR * pairs_per_launch / (k_ms_per / 1e3) / 1e12  # T lane-op/s
    pk_ = peaks()
    sm_max = float(pk_.get("sm_max_mhz", 1965.0))
    peak = 148 * LANES_PER_SM * sm_max * 1e6 / 1e12
    clocks = clk.summary()
    traffic = None
    summ = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if os.path.exists(summ):
        try:
            traffic = json.load(open(summ)).get(cfg.name, {}).get("dram_bytes_per_launch")
        except Exception:
            traffic = None
    kernel_names = {abi.BOIDS_PATH_GRID: "k_grid (binned search + steer + modify)",
                    abi.BOIDS_PATH_SYM: "k_sym (warm-step unordered-pair search)",
                    abi.BOIDS_PATH_SCAN: "k_bound + k_scan (warm-step ordered-pair search)",
                    abi.BOIDS_PATH_THINK: "k_bound + k_scan over this step's thinkers (k_fused for never-searched ones)",
                    abi.BOIDS_PATH_FUSED: "k_fused (cold-step cluster kernel)",
                    abi.BOIDS_PATH_SIMPLE: "k_search_simple (tiled search, thesis structure)",
                    abi.BOIDS_PATH_SMALL: "k_small (whole warm step in one kernel: search + merge + steer + modify)"}
    if sym and dist is not None:
        kernel_names[path] = "k_ss_spbuild + k_sym (this rank's share of the warm-step unordered-pair search)"
    roofline = {"bound": "alu",
                "kernel": kernel_names.get(path, f"path {path}"), "path": path,
                "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak,
                "traffic": traffic,
                "peak_note": f"FP32 SIMT lane-ops: 148 SM x 128 lanes x {sm_max:.0f} MHz "
                             f"(sm_max_mhz of MEASURED_PEAKS.json; each add/sub/mul counted once, no FMA)",
                "work_per_launch": f"{OPS_PER_PAIR} lane-ops x {pairs_per_launch:.4g} pairs" + pairs_note,
                "kernel_ms_per_launch": k_ms_per, "kernel_share_of_step": k_ms / ms if ms else None,
                "timing": ("CUDA events on the launching stream around each search launch of the timed steps"
                           if live else "CUDA events on the launching stream around each search launch of a "
                           "profiled pass of K steps right after the (uninstrumented) timed region"),
                "frac_at_measured_clock": (achieved / (148 * LANES_PER_SM * clocks["sm_mhz"] * 1e6 / 1e12))
                if clocks.get("sm_mhz") else None}
    if sym:  # the thesis's per-agent formulation evaluates n x n ordered pairs
        roofline["ordered_pair_equivalent"] = {
            "achieved": 2 * achieved * cfg.n / (cfg.n - 1) if cfg.n > 1 else 0.0,
            "frac_of_peak": (2 * achieved * cfg.n / (cfg.n - 1) if cfg.n > 1 else 0.0) / peak,
            "note": "n x n pairs of the thesis's formulation / the same kernel time: the rate an "
                    "ordered-pair kernel would need to match; not a hardware utilisation"}

    # ---------------- update and binning kernels against HBM ----------------
    # A separate profiled pass of K steps right after the timed region (events
    # around EVERY launch would break the PDL chain of the timed steps): the
    # update-class kernel (k_select1 on warm brute-force steps, k_apply in think
    # mode) and the binning kernels, each against the measured copy bandwidth.
    # Then the standalone update kernel k_update (B5: steering from the last
    # step's lists + modification, one thread per agent) through
    # boids_bench_update, L2 flushed before every launch.
    hbm = float(pk_.get("hbm_gbs", 6552.0))
    hbm_note = "hbm_gbs of MEASURED_PEAKS.json (copy bandwidth, measured)"
    abi.boids_set_option(h, abi.BOIDS_OPT_PROFILE, 1)
    abi.boids_get_profile(h, reset=True)
    for k in range(args.steps):
        flush.fill_(float(k))
        step()
    torch.cuda.synchronize()
    prof1 = abi.boids_get_profile(h, reset=True)
    abi.boids_set_option(h, abi.BOIDS_OPT_PROFILE, 0)
    u_ms, u_n = prof1["update"]
    update_roofline = None
    if u_n:
        if think > 1 and grid:  # k_apply: pos4 fwd4 up4 side4 fstore in (80 B), pos4 fwd4 up4 side4 out (64 B)
            name, per_agent = "k_apply (modification of every agent, think mode)", 144
        else:  # k_select: ~10 hits (8 B) in, own state in (64 B) / out (64 B); neighbour gathers hit L2
            name, per_agent = "k_select1 (top-7 of the hit buffer + steering + modification)", 128 + 8 * 10
        ub = per_agent * float(nloc) / (u_ms / u_n / 1e3) / 1e9
        update_roofline = {"bound": "hbm", "kernel": name, "achieved": ub, "peak": hbm, "unit": "GB/s",
                           "frac": ub / hbm, "bytes_per_agent": per_agent, "launches": u_n,
                           "kernel_ms_per_launch": u_ms / u_n, "peak_note": hbm_note,
                           "measured": "profiled pass of K steps after the timed region, L2 flushed per step"}
    if sym and dist is None:  # k_sym's prologue (k_sym_prep: warm limits + the ordered SoA copy), timed apart
        p_ms, p_n = prof1["search_prep"]
        s_ms, s_n = prof1["fused_or_search"]
        if p_n and s_n:
            both = p_ms / p_n + s_ms / s_n
            a_both = OPS_PER_PAIR * pairs_per_launch / (both / 1e3) / 1e12
            roofline["prologue"] = {
                "kernel": "k_sym_prep (warm limits, routing, agents in Morton order as SoA)",
                "ms_per_launch": p_ms / p_n,
                "search_incl_prologue": {"kernels": "k_sym_prep + k_sym", "ms_per_launch": both,
                                         "achieved": a_both, "frac": a_both / peak},
                "measured": "profiled pass of K steps after the timed region (events around each launch)"}
    b_ms, b_n = prof1["binning"]
    binning_roofline = None
    if b_n and grid:
        # two binnings per step: candidates by cell -- read pos4 (16), write + read
        # cell/rank (16), read pos4 (16), write the sorted record (16) -- and the owned queries by block --
        # read pos4 (16), write + read cell/rank (16), write the permutation (4); counts amortised
        per_agent = 100
        steps_binned = args.steps
        bb = per_agent * float(cfg.n) * steps_binned / (b_ms / 1e3) / 1e9
        binning_roofline = {"bound": "hbm", "kernel": "k_bin_count + scan + scatter (counting sort by cell)",
                            "achieved": bb, "peak": hbm, "unit": "GB/s", "frac": bb / hbm,
                            "bytes_per_agent": per_agent, "ms_per_step": b_ms / steps_binned,
                            "peak_note": hbm_note}
    std_ms = []
    for k in range(max(3, args.steps)):
        flush.fill_(float(k))
        std_ms.append(abi.boids_bench_update(h, dt, 1))
    std_ms = float(np.median(std_ms))
    per_std = 160  # reads pos4 fwd4 up4 side4 (64) + nbr 7 x 4 + cnt 4 (32); writes pos4 fwd4 up4 side4 (64)
    sb = per_std * float(nloc) / (std_ms / 1e3) / 1e9
    update_standalone = {"bound": "hbm", "kernel": "k_update (steering from the last lists + modification)",
                         "achieved": sb, "peak": hbm, "unit": "GB/s", "frac": sb / hbm,
                         "bytes_per_agent": per_std, "kernel_ms_per_launch": std_ms,
                         "note": "boids_bench_update, median of launches, L2 flushed before each; the "
                                 "neighbours' pos4/fwd4 gathers (up to 7 x 32 B) are not counted (L2 hits)",
                         "peak_note": hbm_note}
    if update_roofline is None:
        update_roofline = dict(update_standalone)

    # ---------------- e2e through the C ABI with host buffers ----------------
    e2e = None
    if args.no_e2e:
        args_e2e = False
    else:
        args_e2e = True
    host = {}
    if args_e2e:  # pinned host arrays (the contract: inputs from pinned host memory)
        for k, shape in (("pos", (nloc, 3)), ("fwd", (nloc, 3)), ("up", (nloc, 3)), ("side", (nloc, 3)),
                         ("speed", (nloc,))):
            host[k] = torch.empty(shape, dtype=torch.float32, pin_memory=True).numpy()
        abi.boids_get_state(h, host)
    h2d = nloc * 13 * 4  # set_state uploads pos3, fwd3, up3, side3, speed (AoS float32)
    d2h = nloc * 13 * 4  # get_state downloads the same
    if args_e2e:
        barrier()
        t0 = time.perf_counter()
        for _ in range(args.steps):
            abi.boids_set_state(h, host)
            step()
            abi.boids_get_state(h, host)
        t1 = time.perf_counter()
        e2e_s = t1 - t0
        if dist is not None:
            t = torch.tensor([e2e_s], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e2e_s = float(t.item())
        e2e = {"value": cfg.n * args.steps / e2e_s, "unit": UNIT, "h2d_bytes_per_step": h2d * world,
               "d2h_bytes_per_step": d2h * world,
               "note": "pinned host AoS arrays: boids_set_state (H2D + device conversion) + step + "
                       "boids_get_state (device conversion + D2H), wall clock"}

    # ---------------- the thesis's draw loop: step + double-buffered readback ----------------
    # (the host consumes step n's 4x4 draw matrices while step n+1 runs)
    e2e_draw = None
    if args_e2e:
        bufs = [torch.empty((nloc, 4, 4), dtype=torch.float32, pin_memory=True).numpy() for _ in range(2)]
        for k in range(2):  # untimed: the copy stream, the first touch of both pinned buffers
            step()
            abi.boids_readback_begin(h, bufs[k % 2])
        abi.boids_readback_wait(h)
        barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for k in range(args.steps):
            step()
            abi.boids_readback_begin(h, bufs[k % 2])
        abi.boids_readback_wait(h)
        e2e_draw_s = time.perf_counter() - t0
        if dist is not None:
            t = torch.tensor([e2e_draw_s], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e2e_draw_s = float(t.item())
        e2e_draw = {"value": cfg.n * args.steps / e2e_draw_s, "unit": UNIT, "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": nloc * 64 * world,
                    "note": "steps with the 4x4 draw matrices (64 B/agent) read back every step on a copy "
                            "stream into alternating pinned buffers (double buffering, P:535-539), wall clock"}

    # ---------------- CPU oracle baseline (rank 0, N=1) ----------------
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        m = cpu_sample_size(cfg, args.cpu_seconds)
        rate, agents, secs = cpu_oracle_rate(cfg, m)
        cpu = {"value": rate, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"{agents} of {cfg.n} agents x 1 step (seeded sample of the config's initial state; "
                         f"each agent a full O(n) search + steer + modify), {secs:.1f} s single-threaded"}
        ncores = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else (os.cpu_count() or 1)
        if ncores > 1:
            r_all, a_all, s_all = cpu_oracle_rate_threads(cfg, max(16, m // 4), ncores)
            cpu["all_cores"] = {"value": r_all, "unit": UNIT, "cores": ncores, "kind": "oracle",
                                "sample": f"{a_all} sampled agents x 1 step split over {ncores} threads, "
                                          f"{s_all:.1f} s"}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": dict(config_dict(cfg, world), think_every=think), "roofline": roofline,
            "update_roofline": update_roofline, "update_standalone": update_standalone,
            "binning_roofline": binning_roofline, "cpu_baseline": cpu, "e2e": e2e, "e2e_draw": e2e_draw,
            "gpu_launches": int(launches), "clocks": clocks,
            "kernel_profile_ms": {k: v[0] for k, v in prof.items() if v[1]},
            "thesis_context": "thesis v5 GPU (GeForce 8800 GTS) vs CPU (Athlon 64 3700+): ~42x at 4096 agents "
                              "(PAPER.md P:499, P:465); different hardware and baseline, not comparable",
        }
        emit(line)
    fl.close()
    if dist is not None:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
