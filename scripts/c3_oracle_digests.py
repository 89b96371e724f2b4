#!/usr/bin/env python
"""Oracle-side expected values for BASELINE config [3] (10^8 traces x 64
containers, config [2] generator) — TEST INFRASTRUCTURE.

Runs the plain C oracle (oracle/oracle_run, single-threaded) on disjoint
2^20-trace ranges in parallel worker processes and records, per policy and
range, the sum of trace digests (mod 2^64) and the range statistics into
tests/golden/c3_range_digests.json.  The file is written incrementally, so a
partial run is still usable (tests compare the ranges that are present).
Only oracle/ computes anything here; the CUDA path is never called.

  python scripts/c3_oracle_digests.py [--workers 7] [--policies 0,1,2,3]
"""
import argparse
import json
import os
import subprocess
import sys
import time
from concurrent.futures import ThreadPoolExecutor, as_completed

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import workloads as W  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "c3_range_digests.json")
RANGE = 1 << 20
POLNAMES = ["fifo", "best_fit", "recent_fit", "random_fit"]


def run_range(w, policy, r):
    g = w.gen
    lo, hi = r * RANGE, min((r + 1) * RANGE, w.n_traces)
    exe = os.path.join(ROOT, "oracle", "oracle_run")
    cmd = [exe, "--n", str(g.n), "--K", str(g.K), "--classes", ",".join(map(str, g.class_mib)),
           "--num", str(g.num), "--den", str(g.den), "--iat", str(g.iat),
           "--gen-seed", str(g.gen_seed), "--dur-base", str(g.dur_base),
           "--dur-step", str(g.dur_step), "--dur-off", str(g.dur_class_offset),
           "--dur-jit", str(g.dur_jit), "--gen-ovh", str(g.ovh), "--ovh", str(w.ovh),
           "--cap", str(w.cap), "--policy", str(policy), "--rand-seed", str(w.rand_seed),
           "--lo", str(lo), "--hi", str(hi), "--range-size", str(RANGE)]
    out = subprocess.run(cmd, capture_output=True, text=True, check=True).stdout
    d = json.loads(out)
    assert len(d["range_digests"]) == 1
    return policy, r, d


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workers", type=int, default=7)
    ap.add_argument("--policies", default="0,1,2,3")
    ap.add_argument("--max-ranges", type=int, default=None)
    args = ap.parse_args()
    oracle.build()
    w = W.CONFIGS["c3"]
    nr = (w.n_traces + RANGE - 1) // RANGE
    if args.max_ranges:
        nr = min(nr, args.max_ranges)
    res = {"citation": "written by scripts/c3_oracle_digests.py from oracle/oracle_run only "
                       "(BASELINE config [3]: workloads.CONFIGS['c3'])",
           "workload": w.name, "n_traces": w.n_traces, "range_size": RANGE, "policies": {}}
    if os.path.exists(OUT):
        with open(OUT) as f:
            res = json.load(f)
    pols = [int(x) for x in args.policies.split(",")]
    jobs = [(p, r) for r in range(nr) for p in pols
            if str(r) not in res["policies"].get(POLNAMES[p], {})]
    print(f"{len(jobs)} ranges to do with {args.workers} workers", flush=True)
    t0 = time.time()
    with ThreadPoolExecutor(args.workers) as ex:
        futs = [ex.submit(run_range, w, p, r) for p, r in jobs]
        for k, f in enumerate(as_completed(futs)):
            p, r, d = f.result()
            ent = res["policies"].setdefault(POLNAMES[p], {})
            ent[str(r)] = {"digest": d["range_digests"][0], "traces": d["traces"],
                           "events": d["events"], "sum_wait": d["sum_wait"],
                           "sum_makespan": d["sum_makespan"], "n_select": d["n_select"],
                           "flag_count": d["flag_count"], "seconds": d["seconds"]}
            tmp = OUT + ".tmp"
            with open(tmp, "w") as fo:
                json.dump(res, fo, indent=0, sort_keys=True)
            os.replace(tmp, OUT)
            print(f"[{k + 1}/{len(jobs)}] {POLNAMES[p]} range {r} "
                  f"{d['seconds']:.0f}s elapsed {time.time() - t0:.0f}s", flush=True)


if __name__ == "__main__":
    main()
