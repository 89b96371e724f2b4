#!/usr/bin/env python
"""bench.py — events replayed per second by the B200 replay of ConVGPU's
GPU-memory scheduler (BASELINE.json metric), one JSON line on rank 0.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

Workload (N=1): BASELINE.json configs[2] — 10^6 traces x 64 containers, 2x
oversubscription of a 180 GiB GPU (workloads.CONFIGS["c2"]).  Rank r replays
global ids [r * 2^20, r * 2^20 + 10^6), so that after the timed steps the
replayed ids plus an untimed tail are exactly 2^20-trace range r of the
oracle's golden file (tests/golden/c3_range_digests.json): every bench run
checks every rank's per-policy digest sum, events, waits, selections and
makespans against the oracle and reports it under "parity" (exit 3 on a
mismatch).  Under torchrun (N>1) this is weak scaling; the per-policy
statistics are all-reduced over NCCL each step and the per-range rows once
after the timed steps.  A "step" = the whole hot path over the batch: replay
under FIFO, Best-Fit, Recent-Fit and Random-Fit (4 launches of the replay
kernel, full per-container outputs + summaries + statistics).  Inputs (2.56
GB per rank) are resident in HBM before the timed region and are larger than
the 126 MB L2, so no flush is needed between steps.  `value` uses the median
step time (median of >= 5 repetitions).

`--workload c3`: BASELINE configs[3] — 10^8 traces sharded [r*N/G, (r+1)*N/G),
chunked generate -> replay on every rank, all 96 golden ranges x 4 policies
checked after an NCCL all-reduce of the range digests (run_c3).

`--impl reference` times the C oracle (test infrastructure, the only
reference this paper-only task has) on the host cores on a bounded sample of
the same workload.
"""
from __future__ import annotations

import argparse
import json
import re
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

METRIC = "scheduler events replayed/sec per policy at 1/2/4/8 B200 (% HBM roofline)"
POLICIES = W.POLICIES


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="c2", choices=["c1", "c2", "c3", "mimic"])
    ap.add_argument("--traces", type=int, default=None, help="traces per GPU (default: config)")
    ap.add_argument("--outputs", default="full", choices=["full", "summary"])
    ap.add_argument("--kernel", default="auto", choices=["auto", "warp", "lane", "lane16"])
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--e2e-chunk", type=int, default=0,
                    help="traces per host-path chunk (0: one full wave of the compact kernel, "
                         "SMs x 256 lanes)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-check", action="store_true", help="skip the golden-range parity check")
    ap.add_argument("--c3-chunk", type=int, default=4 << 20, help="traces per chunk (config [3])")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-sample", type=int, default=32768, help="traces per policy (cpu leg)")
    ap.add_argument("--ref-sample", type=int, default=4096, help="traces per policy per step (reference arm)")
    ap.add_argument("--profile", action="store_true", help="short run for ncu: no sampler/e2e/cpu")
    return ap.parse_args()


def env_rank():
    return (int(os.environ.get("RANK", 0)), int(os.environ.get("LOCAL_RANK", 0)),
            int(os.environ.get("WORLD_SIZE", 1)))


def measured_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


# ------------------------------------------------------------------ clocks
class ClockSampler:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.rows = []
        self.proc = None
        self.thread = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except FileNotFoundError:
            return
        self.thread = threading.Thread(target=self._read, daemon=True)
        self.thread.start()
        time.sleep(0.3)

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.proc is None:
            return None
        time.sleep(0.15)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        self.thread.join(timeout=2)
        sm = [float(r[1]) for r in self.rows if len(r) >= 9 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) >= 9 and r[2].replace(".", "").isdigit()]
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in self.rows:
            if len(r) < 9:
                continue
            for name, v in zip(names, r[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(name)
        loaded = [s for s in sm if s > 0.5 * (max(mx) if mx else 1)] or sm
        return {"sm_mhz": statistics.median(loaded) if loaded else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": sorted(reasons),
                "samples": len(self.rows), "samples_under_load": len(loaded)}


# ------------------------------------------------------------------ oracle timing
def host_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


def oracle_run(w, traces: int, threads: int) -> tuple:
    """Replay global ids [0, traces) under every policy with the C oracle as it
    stands (single-threaded code), on `threads` host threads over disjoint id
    ranges (the ctypes call releases the GIL; every replay keeps its state on
    its own stack).  Returns (events, seconds)."""
    import oracle
    from concurrent.futures import ThreadPoolExecutor
    oracle.build()
    oracle.lib()
    cuts = [traces * j // threads for j in range(threads + 1)]
    jobs = [(p, cuts[j], cuts[j + 1]) for p in POLICIES for j in range(threads) if cuts[j + 1] > cuts[j]]
    run = lambda j: oracle.replay_range(w, j[0], j[1], j[2])["stats"]["events"]  # noqa: E731
    t0 = time.perf_counter()
    if threads == 1:
        ev = sum(run(j) for j in jobs)
    else:
        with ThreadPoolExecutor(threads) as ex:
            ev = sum(ex.map(run, jobs))
    return ev, time.perf_counter() - t0


# ------------------------------------------------------------------ reference arm
def run_reference(args, rank, world):
    """The oracle (plain single-threaded C) timed on this host's cores: one
    oracle thread per core, each on its own slice of the step's traces."""
    if rank != 0:
        return
    w = W.CONFIGS[args.workload]
    C = host_cores()
    S = args.ref_sample * C
    times = []
    events = 0
    for step in range(args.warmup + args.steps):
        ev, dt = oracle_run(w, S, C)
        if step >= args.warmup:
            times.append(dt)
            events += ev
    total = sum(times)
    value = events / total
    sample = (f"{S} traces x {len(POLICIES)} policies per step of {w.name} (ids 0..{S - 1}), "
              f"{C} oracle threads on disjoint id ranges")
    out = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "events/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * total / len(times), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": w.name, "traces_per_step": S, "containers": w.gen.n,
                   "ops_per_container": w.gen.K, "capacity_mib": w.cap,
                   "policies": list(POLICIES)},
        "cpu_baseline": {"value": value, "unit": "events/s", "cores": C, "kind": "oracle",
                         "cpu_model": cpu_model(), "sample": sample},
        "e2e": {"value": value, "unit": "events/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(out), flush=True)


# ------------------------------------------------------------------ our arm
def cpu_baseline(w, sample):
    """The oracle on all host cores (a bounded sample: `sample` traces per core
    and policy), and on one core (`sample` traces per policy)."""
    C = host_cores()
    ev1, dt1 = oracle_run(w, sample, 1)
    evc, dtc = oracle_run(w, sample * C // 2, C)
    return {"value": evc / dtc, "unit": "events/s", "cores": C, "kind": "oracle",
            "cpu_model": cpu_model(),
            "sample": f"{sample * C // 2} traces x {len(POLICIES)} policies of {w.name} "
                      f"(ids 0..{sample * C // 2 - 1}), {C} threads of the single-threaded C "
                      f"oracle on disjoint id ranges, {dtc:.1f} s",
            "single_core": {"value": ev1 / dt1, "cores": 1,
                            "sample": f"{sample} traces x {len(POLICIES)} policies, {dt1:.1f} s"}}


def measured_sm_mhz() -> float:
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return float(json.load(f)["sm_max_mhz"])
    except Exception:
        return 1965.0  # B200 max SM clock (B200_PROFILING.md)


def ncu_summary(workload, traces):
    """DRAM bytes per replay launch and the limiter evidence from the committed
    ncu --set full summary (profiles/ncu_full_summary.json), if it matches."""
    p = os.path.join(ROOT, "profiles", "ncu_full_summary.json")
    try:
        with open(p) as f:
            d = json.load(f)
        if d.get("workload") == workload and int(d.get("traces")) == traces:
            return d
    except Exception:
        pass
    return {}


# ------------------------------------------------------------------ parity
GOLDEN = os.path.join(ROOT, "tests", "golden", "c3_range_digests.json")
RANGE = 1 << 20  # traces per golden range
RANGE_FIELDS = ("digest_sum", "events", "sum_wait", "n_select", "sum_makespan", "traces")


def load_golden(w):
    """Per-2^20-trace-range results of the C oracle for the config [2] / [3]
    generator (tests/golden/c3_range_digests.json, written by
    scripts/c3_oracle_digests.py from oracle/ only; read here as data — no
    oracle code runs).  None if `w` is another workload."""
    c3 = W.CONFIGS["c3"]
    if (w.gen, w.cap, w.ovh, w.rand_seed) != (c3.gen, c3.cap, c3.ovh, c3.rand_seed):
        return None
    try:
        with open(GOLDEN) as f:
            g = json.load(f)
    except OSError:
        return None
    return g if g.get("range_size") == RANGE else None


def golden_row(g, policy, r):
    e = g["policies"].get(policy, {}).get(str(r))
    if e is None:
        return None
    return [int(e["digest"], 16), e["events"], e["sum_wait"], e["n_select"], e["sum_makespan"],
            e["traces"]]


def s64(v: int) -> int:
    v &= (1 << 64) - 1
    return v - (1 << 64) if v >> 63 else v


def stats_row(st) -> list:
    return [st[f] for f in RANGE_FIELDS]


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def max_over_ranks_vec(xs, device, world):
    """Element-wise max over ranks of a list of floats (per-step times)."""
    if world == 1:
        return list(xs)
    import torch
    import torch.distributed as dist
    t = torch.tensor(xs, dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return [float(v) for v in t.cpu()]


SPEC_HBM_GBS = 8000.0  # B200 HBM3e nominal (B200_PROFILING.md), for the "% of spec" figure


def run_ours(args, rank, local_rank, world):
    import torch
    import torch.distributed as dist

    import paper_conf_cluster_kangjkkk17_b200 as cg
    from paper_conf_cluster_kangjkkk17_b200 import dist as cgd

    # one process per GPU; ranks beyond the visible devices share them (only
    # useful with CONVGPU_DIST_BACKEND=gloo, to exercise the N>1 flow on a
    # one-GPU box — NCCL needs one rank per device)
    ndev = torch.cuda.device_count()
    dev = torch.device("cuda", local_rank % ndev)
    torch.cuda.set_device(dev)
    if world > 1:
        backend = os.environ.get("CONVGPU_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    cg.lib()
    if args.workload == "c3":
        return run_c3(args, rank, world, dev, cg, cgd)
    w = W.CONFIGS[args.workload]
    Nr = args.traces or w.n_traces
    n, K = w.gen.n, w.gen.K
    golden = None if args.no_check else load_golden(w)
    if golden is not None and Nr > RANGE:
        golden = None
    # rank r owns global ids [base, base + Nr).  With the config [2] / [3]
    # generator the shard starts at a golden range (base = r * 2^20), so the
    # replayed ids plus an untimed tail are exactly oracle range r.
    base = rank * (RANGE if golden is not None else Nr)
    stream = torch.cuda.current_stream()

    # a0: generation (timed separately, not part of events/s; the first call
    # also loads the module, so time the second)
    tr = cg.generate(w.gen, base, Nr, device=dev)
    g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    g0.record()
    cg.generate(w.gen, base, Nr, device=dev, out=tr)
    g1.record()
    torch.cuda.synchronize()
    gen_ms = g0.elapsed_time(g1)

    full = args.outputs == "full"
    outs = {p: cg.alloc_out(Nr, n, device=dev, full=full, stats=False) for p in POLICIES}
    nsteps = args.warmup + args.steps
    # one [policies, 12] block of convgpu_stats_t records per step
    stats_blk = torch.zeros(nsteps, len(POLICIES), 12, dtype=torch.int64, device=dev)
    stats = {p: stats_blk[:, q] for q, p in enumerate(POLICIES)}
    ev_s = {p: [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)] for p in POLICIES}
    ev_e = {p: [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)] for p in POLICIES}
    step_ev = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps + 1)]

    def step(s, timed_idx=None):
        for p in POLICIES:
            o = outs[p]
            o.stats = stats[p][s]
            if timed_idx is not None:
                ev_s[p][timed_idx].record(stream)
            cg.replay(tr, w.cap, p, o, rand_seed=w.rand_seed, ovh=w.ovh, stream=stream,
                      kernel=args.kernel)
            if timed_idx is not None:
                ev_e[p][timed_idx].record(stream)
        if world > 1:  # the step's exchange: every policy's record, two collectives
            cgd.reduce_stats_block(stats_blk[s])

    for s in range(args.warmup):
        step(s)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    sampler = None
    if not args.profile:
        vis = os.environ.get("CUDA_VISIBLE_DEVICES")
        phys = int(vis.split(",")[dev.index]) if vis else dev.index
        sampler = ClockSampler(phys)
        sampler.start()
    torch.cuda.synchronize()
    step_ev[0].record(stream)
    for k in range(args.steps):
        step(args.warmup + k, k)
        step_ev[k + 1].record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = sampler.stop() if sampler else None
    step_ms = max_over_ranks_vec([step_ev[k].elapsed_time(step_ev[k + 1]) for k in range(args.steps)],
                                 dev, world)
    ms_total = cgd.max_over_ranks(step_ev[0].elapsed_time(step_ev[-1]), dev)
    ms_med = statistics.median(step_ms)

    per_trace_events = n * (1 + K)
    sms = torch.cuda.get_device_properties(dev).multi_processor_count

    def kernel_of(p):  # the rule of abi.cu launch_any / auto_variant
        if args.kernel != "auto":
            return args.kernel
        if Nr < sms * 40:
            return "warp"
        return "lane16" if (n == 64 and K == 4) else "lane"
    launches_per_replay = {p: 3 if kernel_of(p) == "lane16" else 1 for p in POLICIES}
    # correctness of the timed work: every timed launch replayed every trace
    last = args.warmup + args.steps - 1
    checks = {}
    for p in POLICIES:
        st = cg.stats_dict(stats[p][last].cpu().numpy().view(cg.STATS_DTYPE)[0])
        exp_ev = Nr * per_trace_events * world
        assert st["events"] == exp_ev, (p, st["events"], exp_ev)
        assert st["flag_count"] == [0] * 8, (p, st["flag_count"])
        checks[p] = st
    launch_ms = {p: statistics.median(ev_s[p][k].elapsed_time(ev_e[p][k]) for k in range(args.steps))
                 for p in POLICIES}

    events_per_step = world * len(POLICIES) * Nr * per_trace_events
    value = events_per_step / (ms_med / 1e3)

    # parity of the timed work against the oracle (after the timed region):
    # rank r's timed ids + the untimed tail [base + Nr, base + 2^20) form
    # golden range r; per-range rows are SUM-all-reduced (disjoint rows) and
    # rank 0 compares every rank's row with the oracle's
    parity = None
    if golden is not None and not args.profile:
        nt = RANGE - Nr
        rows = {p: torch.zeros(world, len(RANGE_FIELDS), dtype=torch.int64, device=dev) for p in POLICIES}
        tail_st = {p: None for p in POLICIES}
        if nt:
            ttr = cg.generate(w.gen, base + Nr, nt, device=dev)
            for p in POLICIES:
                o = cg.alloc_out(nt, n, device=dev, full=False, summary=False)
                cg.replay(ttr, w.cap, p, o, rand_seed=w.rand_seed, ovh=w.ovh, stream=stream,
                          kernel=args.kernel)
                tail_st[p] = o.stats
            torch.cuda.synchronize()
        # rank r's own row: under N > 1 the timed records were all-reduced in
        # place, so replay rank r's timed ids once more (stats only, same
        # kernel, untimed); at N = 1 that record must equal the timed one
        for p in POLICIES:
            o = cg.alloc_out(Nr, n, device=dev, full=False, summary=False)
            cg.replay(tr, w.cap, p, o, rand_seed=w.rand_seed, ovh=w.ovh, stream=stream,
                      kernel=args.kernel)
            torch.cuda.synchronize()
            own = cg.stats_dict(o.stats_np())
            if world == 1:  # the timed launch's own record must agree
                assert stats_row(own) == stats_row(checks[p]), p
            row = stats_row(own)
            if tail_st[p] is not None:
                t = cg.stats_dict(tail_st[p].cpu().numpy().view(cg.STATS_DTYPE)[0])
                row = [a + b for a, b in zip(row, stats_row(t))]
            rows[p][rank] = torch.tensor([s64(v) for v in row], dtype=torch.int64)
            cgd.reduce_range_digests(rows[p])
        bad = []
        for p in POLICIES:
            got = rows[p].cpu().numpy().astype(np.int64).view(np.uint64)
            for r in range(world):
                want = golden_row(golden, p, r)
                have = [int(v) for v in got[r]]
                if want is None or have != want:
                    bad.append({"policy": p, "range": r, "have": have, "want": want})
        parity = {"ranges": world * len(POLICIES), "equal": not bad,
                  "fields": list(RANGE_FIELDS), "range_size": RANGE,
                  "traces_timed_per_rank": Nr, "tail_traces_per_rank": nt,
                  "source": "tests/golden/c3_range_digests.json (C oracle, scripts/c3_oracle_digests.py)"}
        if bad:
            parity["mismatches"] = bad[:8]

    # roofline of the replay kernel (dominant kernel)
    in_b = n * (2 + 2 * K) * 4
    out_b = (n * 13 if full else 0) + 40
    bytes_per_launch = Nr * (in_b + out_b)
    avg_launch_s = statistics.mean(launch_ms.values()) / 1e3
    peak, peak_src = measured_peak()
    achieved = bytes_per_launch / avg_launch_s / 1e9
    ncu = ncu_summary(w.name, Nr)
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "traffic": ncu.get("dram_bytes_per_launch"),
                "frac_of_spec": achieved / SPEC_HBM_GBS, "spec_peak": SPEC_HBM_GBS,
                "ncu_limiter": ncu.get("limiter"), "ncu_source": ncu.get("source"),
                "kernel": "replay kernels: " + ", ".join(
                    f"{p}={kernel_of(p)}" for p in POLICIES),
                "algorithmic_bytes_per_launch": bytes_per_launch,
                "bytes_per_event": (in_b + out_b) / per_trace_events, "peak_source": peak_src,
                "avg_launch_ms": avg_launch_s * 1e3,
                "note": "HBM is the roofline bound (a few integer ops per byte); the achieved "
                        "rate is limited by each trace's serial event chain (latency / issue), "
                        "see ncu_limiter and DESIGN.md §6.4"}

    # secondary roofline: instruction issue (the binding limit, DESIGN.md
    # §6.4): live events/s x the warp instructions per event of the same
    # kernel in the committed ncu capture, against 4 issue slots per SM per
    # clock (B200: 148 SMs at the measured max SM clock)
    issue = None
    lim = ncu.get("limiter") or {}
    ipe = {}
    for p in POLICIES:
        pid = {"fifo": 0, "best_fit": 1, "recent_fit": 2, "random_fit": 3}[p]
        for kname, v in lim.items():
            # first-pass compact kernel: "<P>" (round 1) or "<P, 0>" (16-bit layout)
            if kernel_of(p) == "lane16" and re.search(rf"replay_lpt16_kernel<{pid}(, (0|false))?>", kname):
                ipe[p] = v
    if len(ipe) == len(POLICIES):
        inst = sum(ipe[p]["warp_instructions_per_event"] * Nr * per_trace_events for p in POLICIES)
        t_s = sum(launch_ms.values()) / 1e3
        sm_mhz = (clocks or {}).get("sm_mhz") or measured_sm_mhz()  # median under load
        peak_issue = sms * 4 * sm_mhz * 1e6
        issue = {"bound": "alu", "achieved": inst / t_s, "peak": peak_issue, "unit": "warp-inst/s",
                 "frac": inst / t_s / peak_issue,
                 "alu_pipe_pct": {p: ipe[p].get("alu_pipe_pct") for p in POLICIES},
                 "warp_execution_efficiency": {p: (ipe[p].get("active_lanes") or 0) / 32.0
                                               for p in POLICIES},
                 "issue_active_pct_ncu": {p: ipe[p].get("issue_active_pct") for p in POLICIES},
                 "source": "ncu warp instructions per event (" + str(ncu.get("source")) + ") x live "
                           "launch times; peak = SMs x 4 schedulers x 1 instr/clk x SM clock under load"}

    result = None
    if rank == 0:
        result = {
            "metric": METRIC, "value": value, "unit": "events/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_med,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "timing": {"value_from": "median over steps of the per-step time (CUDA events on the "
                                     "launching stream, max over ranks)",
                       "step_ms": step_ms, "mean_ms_per_step": ms_total / args.steps,
                       "value_from_mean": events_per_step * args.steps / (ms_total / 1e3)},
            "config": {"workload": w.name + " (BASELINE configs[%s])" % {"c1": 1, "c2": 2}.get(args.workload, "-"),
                       "traces_per_gpu": Nr, "containers": n, "ops_per_container": K,
                       "capacity_mib": w.cap, "policies": list(POLICIES), "outputs": args.outputs,
                       "global_trace_ids": f"[r*{RANGE if golden is not None else Nr}, +{Nr}) per rank r",
                       "l2": "inputs %.2f GB per rank > 126 MB L2; no flush" % (Nr * in_b / 1e9),
                       "parallelism": f"dp{world} (trace-id shards, NCCL stats all-reduce)"},
            "per_policy": {p: {"events_per_s": Nr * per_trace_events * world / (launch_ms[p] / 1e3),
                               "launch_ms": launch_ms[p], "kernel": kernel_of(p),
                               "hbm_frac": bytes_per_launch / (launch_ms[p] / 1e3) / 1e9 / peak,
                               "digest_sum": "%016x" % (checks[p]["digest_sum"] & (2**64 - 1)),
                               "sum_wait": checks[p]["sum_wait"],
                               "sum_makespan": checks[p]["sum_makespan"]} for p in POLICIES},
            "parity": parity,
            "gen_ms": gen_ms,
            "gen_write_gbs": Nr * in_b / (gen_ms / 1e3) / 1e9,
            "roofline": roofline,
            "issue_roofline": issue,
            "gpu_launches": args.steps * sum(launches_per_replay.values()),
            "clocks": clocks,
        }

    # e2e: the same metric through the host-memory C-ABI entry points.  The
    # headline uses the compact 16-bit host format (convgpu_replay_host16: 21
    # B per container instead of 40, unpacked on the device), because the
    # 32-bit path is bound by its PCIe copy; the 32-bit path is timed beside it.
    if not args.no_e2e and not args.profile:
        chunk = args.e2e_chunk or sms * 256  # one trace per lane of a full grid
        t16, oor = cg.pack16(tr, stream=stream)
        torch.cuda.synchronize()
        packed_ok = int(oor.item()) == 0  # every value fits 16 bits (exact)
        h16 = t16.pin() if packed_ok else None
        del t16
        hbuf = [torch.empty(t.shape, dtype=torch.int32, pin_memory=True)
                for t in (tr.arrival, tr.limit, tr.op_delta, tr.op_arg)]
        for h, t in zip(hbuf, (tr.arrival, tr.limit, tr.op_delta, tr.op_arg)):
            h.copy_(t)
        del outs
        torch.cuda.empty_cache()
        hsum_t = torch.empty(len(POLICIES) * Nr * 5, dtype=torch.int64, pin_memory=True)
        hsum = hsum_t.numpy().view(cg.SUMMARY_DTYPE).reshape(len(POLICIES), Nr)
        ws = torch.empty(max(cg.host_workspace_bytes(n, K, chunk, len(POLICIES)),
                             cg.host_workspace_bytes(n, K, chunk, len(POLICIES), packed=True)),
                         dtype=torch.uint8, device=dev)

        def e2e_leg(packed):
            def call():
                if packed:
                    return cg.replay_host16(h16, w.cap, POLICIES, trace_id_base=base,
                                            rand_seed=w.rand_seed, ovh=w.ovh, chunk=chunk,
                                            summary=hsum, workspace=ws, stream=stream,
                                            kernel=args.kernel)
                return cg.replay_host(*hbuf, w.cap, POLICIES, trace_id_base=base,
                                      rand_seed=w.rand_seed, ovh=w.ovh, chunk=chunk,
                                      summary=hsum, workspace=ws, stream=stream, kernel=args.kernel)
            call()  # warm-up
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            times = []
            for _ in range(args.e2e_steps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                st_host = call()
                e1.record(stream)
                torch.cuda.synchronize()
                times.append(e0.elapsed_time(e1))
            times = max_over_ranks_vec(times, dev, world)
            for q, p in enumerate(POLICIES):
                assert int(st_host[q]["events"]) == Nr * per_trace_events
                if rank == 0 and world == 1:
                    assert "%016x" % int(st_host[q]["digest_sum"]) == result["per_policy"][p]["digest_sum"]
            return times

        legs = {}
        if packed_ok:
            legs["u16"] = e2e_leg(True)
        legs["u32"] = e2e_leg(False)
        if rank == 0:
            h2d = {"u16": Nr * n * (2 + 2 + 4 * K + 1), "u32": Nr * in_b}
            api = {"u16": "convgpu_replay_host16 (16-bit host format, unpacked on the device)",
                   "u32": "convgpu_replay_host (32-bit host format)"}
            head = "u16" if packed_ok else "u32"

            def leg_doc(f):
                return {"value": events_per_step / (statistics.median(legs[f]) / 1e3),
                        "unit": "events/s", "steps": args.e2e_steps, "step_ms": legs[f],
                        "h2d_bytes_per_step": h2d[f],
                        "d2h_bytes_per_step": len(POLICIES) * (Nr * 40 + 96),
                        "api": api[f] + ", pinned host buffers, %d-trace chunks, copy/compute "
                                        "overlap" % chunk}
            result["e2e"] = dict(leg_doc(head), outputs=(
                "per-trace 40-B summaries (all fields + digest) and the statistics record per "
                "policy, read back to host each step; per-container outputs are not copied back "
                "(the device-timed `value` writes them to HBM)"))
            result["e2e"]["format"] = head
            if head == "u16":
                result["e2e"]["u32_path"] = leg_doc("u32")
    if rank == 0 and world == 1 and not args.no_cpu_baseline and not args.profile:
        result["cpu_baseline"] = cpu_baseline(w, args.cpu_sample)
    if rank == 0:
        print(json.dumps(result), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    if parity is not None and not parity["equal"]:
        sys.exit(3)


def run_c3(args, rank, world, dev, cg, cgd):
    """BASELINE config [3]: 10^8 traces (config [2] generator) sharded over the
    ranks as contiguous global-id ranges [r*N/G, (r+1)*N/G); each rank cycles
    generate -> replay (4 policies, summary-free: statistics + per-2^20-range
    digests through the admission scratch on the compact kernel) over chunks
    of its range.  After the timed steps the per-range digests and statistics
    are all-reduced (NCCL over NVLink; the only exchange) and rank 0 checks
    all 96 ranges x 4 policies against the oracle's golden digests."""
    import torch
    import torch.distributed as dist

    w = W.CONFIGS["c3"]
    total = args.traces or w.n_traces
    lo, hi = cgd.shard_range(total, rank, world)
    cnt = hi - lo
    n, K = w.gen.n, w.gen.K
    chunk = min(args.c3_chunk, max(cnt, 1))
    nr = (total + RANGE - 1) // RANGE
    stream = torch.cuda.current_stream()
    tr = cg.empty_traces(chunk, n, K, device=dev)
    scratch = torch.empty(chunk, n, dtype=torch.int32, device=dev)
    outs = {}
    for p in POLICIES:
        o = cg.alloc_out(chunk, n, device=dev, full=False, summary=False, range_count=nr,
                         range_size=RANGE, scratch=False)
        o.admit_scratch = scratch
        outs[p] = o
    nchunks = (cnt + chunk - 1) // chunk
    rep_ev = [[(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
               for _ in POLICIES] for _ in range(nchunks)]
    gen_ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
              for _ in range(nchunks)]

    def step(timed):
        for p in POLICIES:
            outs[p].stats.zero_()
            outs[p].range_digest.zero_()
        for j in range(nchunks):
            a = lo + j * chunk
            c = min(chunk, hi - a)
            sub = cg.Traces(tr.arrival[:c], tr.limit[:c], tr.op_delta[:c], tr.op_arg[:c])
            if timed:
                gen_ev[j][0].record(stream)
            cg.generate(w.gen, a, c, out=sub, stream=stream)
            if timed:
                gen_ev[j][1].record(stream)
            for q, p in enumerate(POLICIES):
                if timed:
                    rep_ev[j][q][0].record(stream)
                cg.replay(sub, w.cap, p, outs[p], rand_seed=w.rand_seed, ovh=w.ovh, stream=stream,
                          kernel=args.kernel)
                if timed:
                    rep_ev[j][q][1].record(stream)

    for _ in range(args.warmup):
        step(False)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    vis = os.environ.get("CUDA_VISIBLE_DEVICES")
    phys = int(vis.split(",")[dev.index]) if vis else dev.index
    sampler = None if args.profile else ClockSampler(phys)
    if sampler:
        sampler.start()
    step_ms, rep_ms, gen_ms = [], [], []
    for _ in range(args.steps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        step(True)
        e1.record(stream)
        torch.cuda.synchronize()
        step_ms.append(e0.elapsed_time(e1))
        rep_ms.append(sum(a.elapsed_time(b) for row in rep_ev for a, b in row))
        gen_ms.append(sum(a.elapsed_time(b) for a, b in gen_ev))
    if world > 1:
        dist.barrier()
    clocks = sampler.stop() if sampler else None
    step_ms = max_over_ranks_vec(step_ms, dev, world)
    rep_ms = max_over_ranks_vec(rep_ms, dev, world)
    # the one exchange: statistics + per-range digests of the last step
    for p in POLICIES:
        cgd.reduce_stats(outs[p].stats)
        cgd.reduce_range_digests(outs[p].range_digest)
    torch.cuda.synchronize()
    per_trace_events = n * (1 + K)
    events_per_step = total * per_trace_events * len(POLICIES)
    if rank == 0:
        g = load_golden(w)
        bad, checked = [], 0
        per_policy = {}
        for p in POLICIES:
            st = cg.stats_dict(outs[p].stats_np())
            rd = outs[p].range_digest.cpu().numpy().view(np.uint64)
            tot = [0] * len(RANGE_FIELDS)
            for r in range(nr):
                want = golden_row(g, p, r) if g else None
                if want is None:
                    bad.append({"policy": p, "range": r, "missing": True})
                    continue
                checked += 1
                if int(rd[r]) != want[0]:
                    bad.append({"policy": p, "range": r, "have": "%016x" % int(rd[r]),
                                "want": "%016x" % want[0]})
                tot = [a + b for a, b in zip(tot, want)]
            tot[0] &= (1 << 64) - 1
            have = stats_row(st)
            have[0] &= (1 << 64) - 1
            if total == w.n_traces and have != tot:
                bad.append({"policy": p, "totals": True, "have": have, "want": tot})
            if st["flag_count"] != [0] * 8:
                bad.append({"policy": p, "flags": st["flag_count"]})
            per_policy[p] = {"digest_sum": "%016x" % have[0], "events": st["events"],
                             "sum_wait": st["sum_wait"], "n_select": st["n_select"]}
        ms_med = statistics.median(step_ms)
        result = {
            "metric": METRIC, "value": events_per_step / (ms_med / 1e3), "unit": "events/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_med,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": w.name + " (BASELINE configs[3])", "traces_total": total,
                       "traces_per_gpu": cnt, "chunk_traces": chunk, "containers": n,
                       "ops_per_container": K, "capacity_mib": w.cap, "policies": list(POLICIES),
                       "outputs": "statistics + per-2^20-range digests (summary-free)",
                       "global_trace_ids": "[r*N/G, (r+1)*N/G) per rank r",
                       "step": "generate + replay x 4 policies per chunk, every chunk of the shard",
                       "l2": "inputs %.1f GB per chunk > 126 MB L2; no flush" % (chunk * n * 40 / 1e9),
                       "parallelism": f"dp{world} (trace-id shards, NCCL all-reduce of stats + range digests)"},
            "timing": {"value_from": "median step time incl. on-device generation (max over ranks)",
                       "step_ms": step_ms, "replay_ms": rep_ms,
                       "replay_only_events_per_s": events_per_step / (statistics.median(rep_ms) / 1e3)},
            "per_policy": per_policy,
            "parity": {"ranges": checked, "equal": not bad, "range_size": RANGE,
                       "fields": ["range digest"] + ["totals: " + ",".join(RANGE_FIELDS[1:])],
                       "source": "tests/golden/c3_range_digests.json (C oracle, scripts/c3_oracle_digests.py)",
                       **({"mismatches": bad[:8]} if bad else {})},
            "gpu_launches": args.steps * nchunks * (1 + 3 * len(POLICIES)),
            "clocks": clocks,
        }
        print(json.dumps(result), flush=True)
        ok = not bad
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    if rank == 0 and not ok:  # noqa: F821 (set on rank 0 above)
        sys.exit(3)


def main():
    args = parse()
    rank, local_rank, world = env_rank()
    if world != args.gpus and not (world == 1 and args.gpus == 1):
        if world == 1:
            sys.stderr.write("bench.py: --gpus %d needs torchrun with %d ranks\n" % (args.gpus, args.gpus))
            sys.exit(2)
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    run_ours(args, rank, local_rank, world)


if __name__ == "__main__":
    main()
