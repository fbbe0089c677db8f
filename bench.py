#!/usr/bin/env python
"""bench.py — SYnergy fused predict+select on B200: kernel x frequency evaluations/s.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3] [--impl ours|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...      (one process per GPU, NCCL)

A step = one pass of the whole hot path over one batch: synergy_sweep (model inference for
every (kernel, clock) pair, default-clock normalisation, per-target objectives, masked argmin;
PAPER §6.2) on the rank's kernels, then (N > 1) the NCCL all-gather that assembles
the choice table.  Default workload = BASELINE.json configs[2] (c3: 100 000 kernels x 196 clocks,
500-tree depth-12 forests for speedup and energy, ES/PL targets at 25/50/75 %), the largest
configuration that fits one GPU, per rank, weak scaling (rank r sweeps its own 100 000 kernels of
the seeded population).  Inputs are resident in HBM; L2 is flushed (512 MiB write) between timed
steps (the 65 MB models would otherwise stay in L2).  Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "kernel x frequency evaluations/sec (fused predict+select)"
UNIT = "evals/s"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=50)
    p.add_argument("--warmup", type=int, default=10)
    p.add_argument("--config", default="c3", choices=["c1", "c2", "c3", "c4", "c5"])
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--scaling", default="weak", choices=["weak", "strong"])
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--flush-mib", type=int, default=512)
    p.add_argument("--models", default="rf", choices=["rf", "svr"],
                   help="rf: the config's models (north star); svr: the config's speedup model + an "
                        "SVR_RBF energy model with 512 support vectors (SURVEY NEXT f2)")
    return p.parse_args()


def dist_env():
    return (int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)),
            int(os.environ.get("LOCAL_RANK", 0)))


def bench_models(cfg, which="rf"):
    """(speedup, energy, freqs, default_idx) of the benchmarked workload."""
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    return W.make_models(cfg) if which == "rf" else W.make_models_svr(cfg, n_sv=SVR_SV)


SVR_SV = 512


def workload_desc(cfg, which="rf"):
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    n_k, n_f, sp, en, tg = W.CONFIGS[cfg]
    m = lambda s: "linear" if s[0] == "lin" else f"RF {s[1]}xD{s[2]}"
    tgt = "MAX_PERF,MIN_ENERGY,MIN_EDP,MIN_ED2P,ES_50,PL_50" if tg == "six" else "ES_25,ES_50,ES_75,PL_25,PL_50,PL_75"
    ens = m(en) if which == "rf" else f"SVR_RBF {SVR_SV} SVs"
    return (f"{cfg}{'' if which == 'rf' else '+svr'}: {n_k} kernels x {n_f} core clocks, speedup {m(sp)}, "
            f"energy {ens}, 12 static features, targets {tgt}")


def decisions_per_eval(spec):
    """Internal-node decisions per evaluation of one model (T*D for the complete trees the bench
    configs use; the oracle counts the same quantity)."""
    if spec.forest_weight == 0.0:
        return 0
    import numpy as np
    # depth of each complete BFS tree: nodes = 2^(D+1)-1
    sizes = np.diff(spec.tree_offset)
    return int(sum(int(np.log2(int(s) + 1)) - 1 for s in sizes))


def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as f:
            d = json.load(f)
        return d, "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "sm_max_mhz": 1965.0}, "fallback"


def ncu_traffic(cfg, kernel="k_tm_walk"):
    """dram__bytes_read.sum + dram__bytes_write.sum per launch of `kernel` on `cfg`, from one
    committed ncu --set full capture (profiles/ncu_traffic.json), or None."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(path) as f:
            d = json.load(f).get(cfg, {})
        return d.get(f"{kernel}_dram_bytes_per_launch")
    except Exception:
        return None


def config_dict(cfg, which, world, n_local, flush_mib):
    """The `config` object of the JSON line (identical for our arm and the reference arm)."""
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    n_f = W.CONFIGS[cfg][1]
    sp, en = bench_models(cfg, which)[:2]
    return {"workload": workload_desc(cfg, which), "n_kernels_per_rank": n_local, "n_freqs": n_f,
            "targets": 6, "parallelism": f"dp{world} (kernel axis) + NCCL all-gather of choices",
            "l2": f"flushed between timed steps ({flush_mib} MiB write)",
            "decisions_per_eval": decisions_per_eval(sp) + decisions_per_eval(en)}


# ------------------------------------------------------------------------- clock sampler

class ClockSampler:
    """NVML sampling of SM clock and clocks-event reasons during the timed region."""
    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, device_index, period_s=0.002):
        self.samples, self.reasons_seen = [], set()
        self.max_mhz = None
        self._stop = threading.Event()
        self.period = period_s
        try:
            import pynvml
            pynvml.nvmlInit()
            vis = os.environ.get("CUDA_VISIBLE_DEVICES")
            idx = int(vis.split(",")[device_index]) if vis else device_index
            self.h = pynvml.nvmlDeviceGetHandleByIndex(idx)
            self.nv = pynvml
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.h = None

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                mhz = nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM)
                rs = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                self.samples.append((mhz, rs))
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.h is not None:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        if self.h is not None:
            self._stop.set()
            self._t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unavailable"], "samples": 0}
        load = [(m, r) for m, r in self.samples if not (r & 0x1)] or self.samples
        reasons = set()
        for _, r in load:
            for bit, name in self.REASONS.items():
                if r & bit and bit != 0x1:
                    reasons.add(name)
        return {"sm_mhz": statistics.median(m for m, _ in load), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(reasons), "samples": len(self.samples), "samples_under_load": len(load)}


# -------------------------------------------------------------------------- CPU oracle

def _oracle_range(args):
    cfg, row0, n, models_key = args
    import oracle
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    w = _POOL_CACHE.get(models_key)
    feats = W.make_features(cfg, row0, n)
    t = time.perf_counter()
    oracle.sweep(w[0], w[1], feats, w[2], w[3], w[4])
    return time.perf_counter() - t


_POOL_CACHE = {}


def _pool_init(cfg, which="rf"):
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    import oracle
    oracle.build()
    sp, en, freqs, d = bench_models(cfg, which)
    tg = W.targets_six() if W.CONFIGS[cfg][4] == "six" else W.targets_es_pl()
    _POOL_CACHE[cfg] = (sp, en, freqs, d, tg)


def oracle_single_core(cfg, n_k_cap, budget_s=10.0, which="rf"):
    """The oracle as it stands, one core, on the first kernels of the workload until ~budget_s."""
    import oracle
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    oracle.build()
    w = W.make_config(cfg, row0=0, n=min(n_k_cap, W.CONFIGS[cfg][0]), models=bench_models(cfg, which))
    evals = 0
    t0 = time.perf_counter()
    chunk = max(1, min(w.n_kernels, 100))
    row = 0
    passes = 0
    while True:
        r = oracle.sweep(w.speedup, w.energy, w.features[row:row + chunk], w.freqs, w.default_idx, w.targets)
        evals += r["choice"].shape[0] * w.n_freqs
        row += chunk
        if row >= w.n_kernels:
            row = 0
            passes += 1
        el = time.perf_counter() - t0
        if el >= budget_s and (passes >= 1 or el >= 3 * budget_s):
            break
    return evals / el, evals, el


def run_walk_work(cfg, row0, n_rows, budget=5e8, which="rf"):
    """Run-walk work of the launched rows, counted by the measurement tool tools/workcount.c (not
    the oracle) on the first rows that fit a budget of ~5e8 node decisions (all rows for c1/c2/c5):
    runs of clocks sharing a leaf and their 2-level block fetches."""
    import tools
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    n_f = W.CONFIGS[cfg][1]
    models = bench_models(cfg, which)
    sp, en = models[:2]
    per_row = max(1, n_f * (decisions_per_eval(sp) + decisions_per_eval(en)))
    n = int(min(n_rows, max(16, budget // per_row)))
    if n == 0:
        return None
    w = W.make_config(cfg, row0=row0, n=n, models=models)
    r = tools.count([w.speedup, w.energy], w.features, w.freqs)
    trees = w.speedup.n_trees + w.energy.n_trees
    return {"run_blocks_per_kernel": r["run_blocks"] / n, "resume_blocks_per_kernel": r["resume_blocks"] / n,
            "runs_per_kernel_tree": r["runs"] / (n * max(trees, 1)),
            "sample": f"rows [{row0}, {row0 + n}) of {cfg}" + (" (all launched rows)" if n == n_rows else
                                                             f" scaled to {n_rows} rows")}


def run_reference(args, rank, world):
    """Reference arm: the CPU oracle (as it stands, single-threaded per process) on the box's host
    cores, one process per core over contiguous kernel ranges of a bounded sample per step."""
    if rank != 0:
        return
    import multiprocessing as mp
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    cfg = args.config
    n_k, n_f = W.CONFIGS[cfg][0], W.CONFIGS[cfg][1]
    cores = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else os.cpu_count()
    sp, en, freqs, d = bench_models(cfg, args.models)
    dec = decisions_per_eval(sp) + decisions_per_eval(en)
    # bounded sample: ~2 s of wall per step at ~6e7 decisions/s/core (calibrated below)
    ctx = mp.get_context("fork")
    with ctx.Pool(cores, initializer=_pool_init, initargs=(cfg, args.models)) as pool:
        t = pool.map(_oracle_range, [(cfg, 0, 1, cfg)] * cores)
        per_kernel = max(min(t), 1e-4)
        sample = int(max(cores, min(n_k, 2.0 / per_kernel * cores)))
        per = (sample + cores - 1) // cores
        jobs = [(cfg, i * per, min(per, sample - i * per), cfg) for i in range(cores) if i * per < sample]
        for _ in range(args.warmup):
            pool.map(_oracle_range, jobs)
        times = []
        for _ in range(args.steps):
            t0 = time.perf_counter()
            pool.map(_oracle_range, jobs)
            times.append(time.perf_counter() - t0)
    ms = 1e3 * sum(times) / len(times)
    value = sample * n_f / (sum(times) / len(times))
    desc = f"first {sample} kernels of {cfg} per step, {len(jobs)} processes x single-threaded oracle"
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": args.scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": config_dict(cfg, args.models, world, n_k if args.scaling == "weak" else -(-n_k // world),
                                  args.flush_mib),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": len(jobs), "kind": "oracle", "sample": desc,
                             "sample_kernels_per_step": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------ ours

def main():
    args = parse()
    rank, world, local = dist_env()
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    import numpy as np
    import torch
    import torch.distributed as dist

    from paper_conf_sc_fandccfc23_b200 import build as B
    from paper_conf_sc_fandccfc23_b200 import synergy as syn
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    from paper_conf_sc_fandccfc23_b200.dist import ShardedSweep, shard_rows

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        import datetime
        dist.init_process_group("nccl", device_id=dev, timeout=datetime.timedelta(seconds=600))
    if rank == 0:
        B.build()
    if world > 1:
        dist.barrier()
    syn.load()

    cfg = args.config
    n_cfg, n_f = W.CONFIGS[cfg][0], W.CONFIGS[cfg][1]
    sp_spec, en_spec, freqs, d = bench_models(cfg, args.models)
    targets = W.targets_six() if W.CONFIGS[cfg][4] == "six" else W.targets_es_pl()
    weak = args.scaling == "weak"
    if weak:
        row0, n_local = rank * n_cfg, n_cfg
    else:
        row0, n_local, _ = shard_rows(n_cfg, rank, world)
    feats_np = W.make_features(cfg, row0, n_local)
    sp, en, ck = syn.Model(sp_spec, local), syn.Model(en_spec, local), syn.Clocks(freqs, local)
    feats = torch.from_numpy(feats_np).to(dev)
    n_t = len(targets)
    sharded = ShardedSweep(n_cfg, n_t, rank, world, dev, weak=weak,
                           compute=lambda f, o: syn.sweep(sp, en, f, ck, d, targets, out=o))
    flush = torch.empty(args.flush_mib * (1 << 20) // 4, dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream()

    def step():
        return sharded.run(feats)

    # warm-up (untimed), incl. a short clock ramp so the timed region runs at load clocks
    for _ in range(args.warmup):
        flush.zero_()
        step()
    t_end = time.time() + 0.5
    while time.time() < t_end:          # bounded: one step in flight at a time
        step()
        torch.cuda.synchronize()

    K = args.steps
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True),
           torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    launches = 0
    sampler = ClockSampler(local)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with sampler:
        for i in range(K):
            flush.zero_()                                   # L2 flush, outside the events
            ev[i][0].record(stream)
            if sharded.n_local:
                syn.sweep(sp, en, feats, ck, d, targets, out=sharded.local[:sharded.n_local])
                launches += syn.last_launch()["kernels"]
            ev[i][1].record(stream)
            if world > 1:
                dist.all_gather_into_tensor(sharded.table, sharded.local)
            ev[i][2].record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
    # Per-kernel times for the roofline come from a second pass of K steps with the library's
    # per-launch events on (they add ~10 us per step on c2, so they stay out of the timed region).
    syn.timing_read()                                       # drop anything recorded so far
    syn.timing_enable(True)                                 # per-kernel events on the launch stream
    evk = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    for i in range(K):
        flush.zero_()
        evk[i][0].record(stream)
        if sharded.n_local:
            syn.sweep(sp, en, feats, ck, d, targets, out=sharded.local[:sharded.n_local])
        evk[i][1].record(stream)
    torch.cuda.synchronize()
    syn.timing_enable(False)
    ktimes = syn.timing_read()                              # {kernel: (total ms, launches, busy ms)}
    ktimed_ms = sum(a.elapsed_time(b) for a, b in evk)      # the instrumented pass's own steps
    kern_ms = [a.elapsed_time(b) for a, b, _ in ev]
    step_ms = [a.elapsed_time(c) for a, _, c in ev]
    total_ms = sum(step_ms)
    tot = torch.tensor([total_ms, sum(kern_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.MAX)
    total_ms_max = float(tot[0])
    evals_step = (n_local if not weak else n_cfg) * n_f
    evals_all = (n_cfg * world if weak else n_cfg) * n_f
    value = evals_all * K / (total_ms_max / 1e3)

    # ------------------------------------------------ e2e through the host-buffer C-ABI path
    e2e = None
    if not args.no_e2e:
        h_feats = torch.from_numpy(feats_np).pin_memory()
        e_ms = []
        if world == 1:
            ws = syn.Workspace(local)
            h_out = torch.empty((n_local, n_t), dtype=torch.int32).pin_memory()
            for i in range(args.warmup + K):
                flush.zero_()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                ws.sweep_host(sp, en, h_feats, ck, d, targets, h_out)
                b.record(stream)
                b.synchronize()
                if i >= args.warmup:
                    e_ms.append(a.elapsed_time(b))
            h2d, d2h = h_feats.numel() * 4, h_out.numel() * 4
            ref_ok = bool((h_out.to(dev) == sharded.local[:n_local]).all())
        else:
            d_feats = torch.empty_like(feats)
            h_table = torch.empty(tuple(sharded.gathered().shape), dtype=torch.int32).pin_memory()
            for i in range(args.warmup + K):
                flush.zero_()
                dist.barrier()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                d_feats.copy_(h_feats, non_blocking=True)
                tbl = sharded.run(d_feats)
                h_table.copy_(tbl, non_blocking=True)
                b.record(stream)
                b.synchronize()
                if i >= args.warmup:
                    e_ms.append(a.elapsed_time(b))
            h2d, d2h = h_feats.numel() * 4, h_table.numel() * 4
            ref_ok = True
        et = torch.tensor([sum(e_ms)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(et, op=dist.ReduceOp.MAX)
        e2e = {"value": evals_all * K / (float(et[0]) / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
               "ms_per_step": float(et[0]) / K, "matches_device_path": ref_ok}

    # ------------------------------------------------------------------------- roofline
    peaks, peak_src = load_peaks()
    sms = torch.cuda.get_device_properties(dev).multi_processor_count
    sm_max = float(peaks.get("sm_max_mhz", 1965.0))
    dec = decisions_per_eval(sp_spec) + decisions_per_eval(en_spec)
    # dominant kernel of the step, timed by the library's events on its launch stream
    algo = max(ktimes, key=lambda k: ktimes[k][2]) if ktimes else "k_tm_walk"
    # the kernel's time per launch: the union of its launch intervals / launches (the slab
    # pipeline's walks alternate between two streams and overlap, so the mean launch duration
    # would count the overlap twice); equal to the mean duration when launches do not overlap
    kern_avg_s = (ktimes[algo][2] / ktimes[algo][1] / 1e3) if ktimes else statistics.mean(kern_ms) / 1e3
    kernel_share = ktimes[algo][2] / ktimed_ms if ktimes else sum(kern_ms) / total_ms
    per_kernel = {k: {"ms_per_launch": v[0] / v[1], "busy_ms_per_launch": v[2] / v[1], "launches": v[1],
                      "share_of_step": v[2] / ktimed_ms}
                  for k, v in ktimes.items()}
    hbm_bytes = evals_step // n_f * (W.N_STATIC * 4 + n_t * 4) + n_f * 4 + \
        sp.info()["device_bytes"] + en.info()["device_bytes"]
    hbm_ach = hbm_bytes / kern_avg_s / 1e9
    hbm = {"achieved": hbm_ach, "peak": peaks["hbm_gbs"], "unit": "GB/s", "frac": hbm_ach / peaks["hbm_gbs"],
           "algorithmic_bytes": hbm_bytes, "peak_source": peak_src}
    # on-chip ceilings measured on this GPU now (tools/peaks.cu): scattered 32-byte L1-resident
    # loads (the k_tm_walk block fetch), the same from L2, conflict-free shared-memory reads
    import tools
    try:
        onchip = tools.measure_peaks(local)
    except Exception as exc:                                       # noqa: BLE001
        onchip = {"error": str(exc)}
    work = None
    if rank == 0 and algo == "k_tm_walk":
        work = run_walk_work(cfg, row0, n_local, which=args.models)
    if algo == "k_svr":
        # fp64 FMA-pipe roofline: 2 * n_k * n_f * n_SV flops per contraction
        per_step = max(1.0, ktimes[algo][1] / K)              # kernel-slab launches per step
        flops = 2.0 * (evals_step // n_f) * n_f * en_spec.n_sv / per_step
        achieved = flops / kern_avg_s / 1e12
        peak = 64 * 2 * sms * sm_max * 1e6 / 1e12
        roofline = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak,
                    "traffic": None, "kernel": algo, "kernel_ms": kern_avg_s * 1e3, "kernel_time": "busy (union of launch intervals) per launch",
                    "kernel_share_of_step": kernel_share, "algorithmic_flops_per_launch": flops,
                    "peak_note": f"fp64 FMA pipe 64 FMA/clk/SM x 2 x {sms} SMs x {sm_max:.0f} MHz (derived; "
                                 "tcgen05 has no fp64 kind)",
                    "hbm": hbm, "per_kernel": per_kernel}
    elif work is not None and "l1_scatter32_bytes_per_s" in onchip:
        # on-chip L1 roofline: each resume walk fetches 32-byte 2-level blocks;
        # counted by tools/workcount.c from the inputs; peak = the measured rate of exactly that
        # access (independent scattered 256-bit loads hitting L1) on this GPU
        per_launch = max(1.0, ktimes[algo][1] / K)             # kernel-slab launches per step
        blocks = work["resume_blocks_per_kernel"] * (evals_step // n_f) / per_launch
        achieved = 32.0 * blocks / kern_avg_s / 1e9
        peak = onchip["l1_scatter32_bytes_per_s"] / 1e9
        roofline = {"bound": "l1", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                    "peak_source": "measured (tools/peaks.cu k_scatter32 on this GPU in this run)",
                    "traffic": ncu_traffic(cfg, algo) if args.models == "rf" else None, "kernel": algo,
                    "kernel_ms": kern_avg_s * 1e3, "kernel_time": "busy (union of launch intervals) per launch", "kernel_share_of_step": kernel_share,
                    "algorithmic_bytes_per_launch": 32.0 * blocks,
                    "work": {"unit": "32-byte 2-level block fetches of the resume walks (each run restarts "
                                     "where its path leaves the previous run's)",
                             "per_launch": blocks,
                             "runs_per_kernel_tree": work["runs_per_kernel_tree"], "counted_on": work["sample"]},
                    "onchip_peaks_measured": onchip,
                    "nominal_l1_bytes_per_s": 128.0 * sms * sm_max * 1e6,
                    "decisions_per_s_vs_direct": evals_step * dec / kern_avg_s,
                    "hbm": hbm, "per_kernel": per_kernel}
    else:
        achieved = evals_step * dec / kern_avg_s / 1e9                  # G node-decisions / s
        peak = sms * sm_max * 1e6 * 32 / 2 / 1e9
        roofline = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Gdecisions/s",
                    "frac": achieved / peak, "traffic": ncu_traffic(cfg, algo) if args.models == "rf" else None,
                    "kernel": algo, "kernel_ms": kern_avg_s * 1e3, "kernel_time": "busy (union of launch intervals) per launch", "kernel_share_of_step": kernel_share,
                    "peak_note": f"{sms} SMs x {sm_max:.0f} MHz x 32 lanes / 2 L1 wavefronts per decision (derived)",
                    "onchip_peaks_measured": onchip, "hbm": hbm, "per_kernel": per_kernel}

    if "k_svr_tc" in ktimes:
        # the SVR contraction on tcgen05: the int8 digit products it issues (28 digit pairs x
        # 2 * M * N * K per tile, padded tiles) against the int8 dense peak (measured bf16 x 2, the
        # nominal int8 / bf16 ratio 4.5 / 2.25 PFLOP/s)
        tc_s = ktimes["k_svr_tc"][0] / ktimes["k_svr_tc"][1] / 1e3
        per_step = max(1.0, ktimes["k_svr_tc"][1] / K)
        n_k_l = evals_step // n_f
        n_svp = -(-en_spec.n_sv // 32) * 32
        tc_n = 32                                           # kTcN: clocks per k_svr_tc tile (kernels_svr_tc.cuh)
        ops = 28 * 2.0 * (-(-n_k_l // 128) * 128) * (-(-n_f // tc_n) * tc_n) * n_svp / per_step
        roofline["svr_contraction"] = {
            "bound": "tensor", "kernel": "k_svr_tc", "kernel_ms": tc_s * 1e3, "achieved": ops / tc_s / 1e12,
            "peak": 2.0 * peaks["bf16_tflops"], "unit": "TOP/s (int8)",
            "frac": ops / tc_s / 1e12 / (2.0 * peaks["bf16_tflops"]), "int8_ops_per_launch": ops,
            "fp64_equivalent_tflops": 2.0 * n_k_l * n_f * en_spec.n_sv / per_step / tc_s / 1e12,
            "peak_note": f"int8 dense = 2 x measured bf16 {peaks['bf16_tflops']} TFLOP/s ({peak_src})"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        v, ev_n, el = oracle_single_core(cfg, min(n_cfg, 1000), which=args.models)
        cpu = {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"first {min(n_cfg, 1000)} kernels of {cfg} x {n_f} clocks repeated to "
                         f"{el:.1f} s ({ev_n} evals), single-threaded oracle (oracle/oracle.c)"}

    if rank == 0:
        clocks = sampler.summary()
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K,
                "warmup": args.warmup, "ms_per_step": total_ms_max / K, "higher_is_better": True,
                "scaling": args.scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": config_dict(cfg, args.models, world, n_local, args.flush_mib),
                "gpu_launches": launches, "roofline": roofline, "e2e": e2e, "cpu_baseline": cpu,
                "clocks": clocks}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
