#!/usr/bin/env python
"""BASELINE config [4]: capacity / oversubscription sweep on the 180 GiB model.

For rho = 1..8 (declared limits scaled by 15*rho/7, so E[sum L]/cap = rho),
10^6 traces x 64 containers per point, Random-Fit replayed with seeds
0..31 and FIFO / Best-Fit / Recent-Fit once, all on the GPU through the C ABI
(statistics only, no per-trace outputs).  Writes per-(rho, policy, seed) means
and the seed spread to profiles/<tag>_rho_sweep.json and a markdown table.

  python scripts/rho_sweep.py [--traces 1000000] [--seeds 32] [--lit-seeds 8] [--rhos 1-8] [--tag r02]

NEXT-1: every point is also replayed under the literal
re-select-on-every-release reading R1-LIT (warp-per-trace kernel), all four
policies (Random-Fit seeds 0..lit_seeds-1), recording the deadlock share per
policy and rho (the paper's no-deadlock claim, P:7, under the other reading)
and the means over the traces that did not deadlock.

Under torchrun (G ranks, one per GPU) every point's trace-id range [0, N) is
sharded [r*N/G, (r+1)*N/G): each rank generates and replays its own shard and
the per-run statistics record is all-reduced (dist.reduce_stats: NCCL SUM /
MAX), so the table is identical for any G (tests/test_gpu_dist.py checks the
digest sums of 1 vs 2 ranks); replay time per run is the max over ranks.

  python -m torch.distributed.run --nproc-per-node 8 --master-addr 127.0.0.1 scripts/rho_sweep.py

Parity of the sweep's kernels against the oracle is covered by
tests/test_gpu_parity.py::test_rho_sweep_window and tests/test_gpu_lane16.py.
"""
import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--traces", type=int, default=1_000_000)
    ap.add_argument("--seeds", type=int, default=32)
    ap.add_argument("--lit-seeds", type=int, default=8)
    ap.add_argument("--rhos", default="1-8", help="e.g. 1-8 or 2,8")
    ap.add_argument("--tag", default="r02")
    ap.add_argument("--out", default=None, help="output JSON (default gpurun_out/ or profiles/)")
    a = ap.parse_args()
    lo_r, _, hi_r = a.rhos.partition("-")
    rhos = list(range(int(lo_r), int(hi_r) + 1)) if hi_r else [int(x) for x in a.rhos.split(",")]
    import torch
    import torch.distributed as dist

    import paper_conf_cluster_kangjkkk17_b200 as cg
    from paper_conf_cluster_kangjkkk17_b200 import dist as cgd
    # one process per GPU under torchrun (ranks beyond the visible devices
    # share them; CONVGPU_DIST_BACKEND=gloo for that case)
    rank, world = int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    dev = torch.device("cuda", local % torch.cuda.device_count())
    torch.cuda.set_device(dev)
    if world > 1:
        backend = os.environ.get("CONVGPU_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    # every point's trace ids [0, traces) are sharded [r*N/G, (r+1)*N/G)
    t_lo, t_hi = cgd.shard_range(a.traces, rank, world)
    cnt = t_hi - t_lo

    def run(w, buf, pol, seed):
        """Replay this rank's shard; statistics all-reduced over the ranks
        (NCCL: SUM / MAX on the 96-B record), time = max over ranks."""
        out = cg.alloc_out(cnt, w.gen.n, device=dev, full=False, summary=False)
        # limits above 0xFFFE MiB (rho = 8): the compact kernel's 17-bit
        # layout first (R1; every such trace would take its second pass)
        wide = max(w.gen.class_mib) * w.gen.num // w.gen.den > 0xFFFE and "literal" not in pol
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        cg.replay(buf, w.cap, pol, out, rand_seed=seed, kernel="lane16w" if wide else "auto")
        e1.record()
        torch.cuda.synchronize()
        ms = cgd.max_over_ranks(e0.elapsed_time(e1), dev)
        cgd.reduce_stats(out.stats)
        st = cg.stats_dict(out.stats_np())
        assert st["traces"] == a.traces, (st["traces"], a.traces)
        return st, ms

    # untimed warm-up: the first launch of each kernel loads its module (lazy
    # loading), which must not land in the first point's time
    for rho in (rhos[0], rhos[-1]):
        w = W.rho_sweep(rho, n_traces=a.traces)
        wb = cg.generate(w.gen, t_lo, min(cnt, 8192), device=dev)
        for pol in ("fifo", "best_fit", "recent_fit", "random_fit"):
            for p in (pol, pol + "+literal"):
                cg.replay(wb, w.cap, p, cg.alloc_out(wb.count, w.gen.n, device=dev, full=False,
                                                     summary=False),
                          kernel="lane16w" if (max(w.gen.class_mib) * w.gen.num // w.gen.den > 0xFFFE
                                               and "literal" not in p) else "lane16")
    torch.cuda.synchronize()
    rows = []
    t_all = time.time()
    buf = None
    for rho in rhos:
        w = W.rho_sweep(rho, n_traces=a.traces)
        buf = cg.generate(w.gen, t_lo, cnt, device=dev, out=buf)
        runs = [("fifo", 0), ("best_fit", 0), ("recent_fit", 0)] + \
               [("random_fit", s) for s in range(a.seeds)]
        for pol, seed in runs:
            st, ms = run(w, buf, pol, seed)
            rows.append({"rho": rho, "policy": pol, "seed": seed,
                         "mean_makespan_s": st["sum_makespan"] / st["traces"] / 1000.0,
                         "mean_wait_s": st["sum_wait"] / (st["traces"] * w.gen.n) / 1000.0,
                         "selections_per_trace": st["n_select"] / st["traces"],
                         "max_peak_reserved_mib": st["max_peak_reserved"],
                         "flag_count": st["flag_count"], "digest_sum": "%016x" % st["digest_sum"],
                         "events": st["events"], "ms": ms})
    # R1-LIT (NEXT-1): deadlock share per policy and rho
    lit_rows = []
    for rho in rhos:
        w = W.rho_sweep(rho, n_traces=a.traces)
        buf = cg.generate(w.gen, t_lo, cnt, device=dev, out=buf)
        runs = [("fifo", 0), ("best_fit", 0), ("recent_fit", 0)] + \
               [("random_fit", s) for s in range(a.lit_seeds)]
        for pol, seed in runs:
            st, ms = run(w, buf, pol + "+literal", seed)
            ok = st["traces"] - st["flag_count"][0]  # deadlocked traces report zeros
            lit_rows.append({"rho": rho, "policy": pol, "seed": seed,
                             "deadlock_share": st["flag_count"][0] / st["traces"],
                             "mean_makespan_s_ok": st["sum_makespan"] / max(ok, 1) / 1000.0,
                             "mean_wait_s_ok": st["sum_wait"] / (max(ok, 1) * w.gen.n) / 1000.0,
                             "digest_sum": "%016x" % st["digest_sum"], "events": st["events"],
                             "ms": ms})
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    if rank != 0:
        return
    lit_table = []
    for rho in rhos:
        line = {"rho": rho}
        for pol in ("fifo", "best_fit", "recent_fit", "random_fit"):
            rr = [x for x in lit_rows if x["rho"] == rho and x["policy"] == pol]
            line[pol] = {"deadlock_share": statistics.mean(x["deadlock_share"] for x in rr),
                         "mean_makespan_s_ok": statistics.mean(x["mean_makespan_s_ok"] for x in rr),
                         "mean_wait_s_ok": statistics.mean(x["mean_wait_s_ok"] for x in rr)}
        lit_table.append(line)
    table = []
    for rho in rhos:
        line = {"rho": rho}
        for pol in ("fifo", "best_fit", "recent_fit"):
            r = [x for x in rows if x["rho"] == rho and x["policy"] == pol][0]
            line[pol] = (r["mean_makespan_s"], r["mean_wait_s"])
        rr = [x for x in rows if x["rho"] == rho and x["policy"] == "random_fit"]
        mk = [x["mean_makespan_s"] for x in rr]
        wt = [x["mean_wait_s"] for x in rr]
        line["random_fit"] = {"makespan_mean": statistics.mean(mk),
                              "makespan_sd": statistics.pstdev(mk),
                              "makespan_min": min(mk), "makespan_max": max(mk),
                              "wait_mean": statistics.mean(wt), "wait_sd": statistics.pstdev(wt)}
        line["deadlocks"] = sum(x["flag_count"][0] for x in rows if x["rho"] == rho)
        table.append(line)
    ev = sum(x["events"] for x in rows)
    ms = sum(x["ms"] for x in rows)
    doc = {"config": "BASELINE configs[4]", "traces_per_point": a.traces, "seeds": a.seeds,
           "n_gpus": world, "sharding": "trace ids [r*N/G, (r+1)*N/G) per rank; stats all-reduced",
           "time": "per run: CUDA events around the replay launch, max over ranks",
           "capacity_mib": 184320, "containers": 64, "unit_time": "s (1 tick = 1 ms)",
           "replay_events": ev, "replay_ms": ms, "events_per_s": ev / (ms / 1e3),
           "wall_s": time.time() - t_all, "table": table, "runs": rows,
           "literal": {"reading": "R1-LIT (DESIGN.md §6.5, NEXT-1)", "seeds": a.lit_seeds,
                       "events": sum(x["events"] for x in lit_rows),
                       "events_per_s": sum(x["events"] for x in lit_rows) /
                       (sum(x["ms"] for x in lit_rows) / 1e3),
                       "table": lit_table, "runs": lit_rows}}
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    path = a.out or (os.path.join(ROOT, "gpurun_out", f"{a.tag}_rho_sweep.json")
                     if os.path.isdir(os.path.join(ROOT, "gpurun_out")) else
                     os.path.join(ROOT, "profiles", f"{a.tag}_rho_sweep.json"))
    with open(path, "w") as f:
        json.dump(doc, f, indent=1)
    print("rho | FIFO makespan/wait | BF | RU | Rand makespan mean±sd [min,max] / wait | deadlocks")
    for l in table:
        r = l["random_fit"]
        print(f"{l['rho']} | {l['fifo'][0]:.1f}/{l['fifo'][1]:.1f} | {l['best_fit'][0]:.1f}/"
              f"{l['best_fit'][1]:.1f} | {l['recent_fit'][0]:.1f}/{l['recent_fit'][1]:.1f} | "
              f"{r['makespan_mean']:.2f}±{r['makespan_sd']:.3f} [{r['makespan_min']:.2f},"
              f"{r['makespan_max']:.2f}] / {r['wait_mean']:.2f} | {l['deadlocks']}")
    print(f"{ev:.3e} events in {ms / 1e3:.2f} s of replay = {ev / (ms / 1e3):.3e} events/s")
    print("R1-LIT deadlock share: rho | FIFO | BF | RU | Rand")
    for l in lit_table:
        print(f"{l['rho']} | " + " | ".join(f"{l[p]['deadlock_share']:.4f}" for p in
                                            ("fifo", "best_fit", "recent_fit", "random_fit")))


if __name__ == "__main__":
    main()
