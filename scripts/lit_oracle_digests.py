#!/usr/bin/env python
"""Oracle-side expected values for R1-LIT (NEXT-1) at scale — TEST
INFRASTRUCTURE.  Runs the plain C oracle (oracle/oracle_run,
single-threaded) under the literal reading on 2^20-trace ranges of config
[4] at ρ = 3 and 5 (where the literal reading deadlocks part of the traces
under Random-Fit) and records per (ρ, policy, range) the sum of trace
digests and the range statistics into tests/golden/lit_range_digests.json.
Only oracle/ computes anything here; the CUDA path is never called.

  python scripts/lit_oracle_digests.py [--workers 8] [--ranges 2]
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

OUT = os.path.join(ROOT, "tests", "golden", "lit_range_digests.json")
RANGE = 1 << 20
POLNAMES = ["fifo", "best_fit", "recent_fit", "random_fit"]
LITERAL = 0x100
RHOS = (3, 5)
RAND_SEED = 11


def run_range(rho, policy, r):
    w = W.rho_sweep(rho, n_traces=(r + 1) * RANGE, rand_seed=RAND_SEED)
    g = w.gen
    lo, hi = r * RANGE, (r + 1) * RANGE
    exe = os.path.join(ROOT, "oracle", "oracle_run")
    cmd = [exe, "--n", str(g.n), "--K", str(g.K), "--classes", ",".join(map(str, g.class_mib)),
           "--num", str(g.num), "--den", str(g.den), "--iat", str(g.iat),
           "--gen-seed", str(g.gen_seed), "--dur-base", str(g.dur_base),
           "--dur-step", str(g.dur_step), "--dur-off", str(g.dur_class_offset),
           "--dur-jit", str(g.dur_jit), "--gen-ovh", str(g.ovh), "--ovh", str(w.ovh),
           "--cap", str(w.cap), "--policy", str(policy | LITERAL), "--rand-seed", str(RAND_SEED),
           "--lo", str(lo), "--hi", str(hi), "--range-size", str(RANGE)]
    out = subprocess.run(cmd, capture_output=True, text=True, check=True).stdout
    d = json.loads(out)
    assert len(d["range_digests"]) == 1
    return rho, policy, r, d


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workers", type=int, default=8)
    ap.add_argument("--ranges", type=int, default=2)
    args = ap.parse_args()
    oracle.build()
    res = {"citation": "written by scripts/lit_oracle_digests.py from oracle/oracle_run only "
                       "(R1-LIT, BASELINE config [4] generator: workloads.rho_sweep(rho))",
           "range_size": RANGE, "rand_seed": RAND_SEED, "rhos": {}}
    if os.path.exists(OUT):
        with open(OUT) as f:
            res = json.load(f)
    jobs = [(rho, p, r) for rho in RHOS for p in range(4) for r in range(args.ranges)
            if str(r) not in res["rhos"].get(str(rho), {}).get(POLNAMES[p], {})]
    print(f"{len(jobs)} ranges to do with {args.workers} workers", flush=True)
    t0 = time.time()
    with ThreadPoolExecutor(args.workers) as ex:
        futs = [ex.submit(run_range, *j) for j in jobs]
        for k, f in enumerate(as_completed(futs)):
            rho, p, r, d = f.result()
            ent = res["rhos"].setdefault(str(rho), {}).setdefault(POLNAMES[p], {})
            ent[str(r)] = {"digest": d["range_digests"][0], "traces": d["traces"],
                           "events": d["events"], "sum_wait": d["sum_wait"],
                           "sum_makespan": d["sum_makespan"], "n_select": d["n_select"],
                           "flag_count": d["flag_count"], "seconds": d["seconds"]}
            tmp = OUT + ".tmp"
            with open(tmp, "w") as fo:
                json.dump(res, fo, indent=0, sort_keys=True)
            os.replace(tmp, OUT)
            print(f"[{k + 1}/{len(jobs)}] rho {rho} {POLNAMES[p]} range {r} "
                  f"{d['seconds']:.0f}s elapsed {time.time() - t0:.0f}s", flush=True)


if __name__ == "__main__":
    main()
