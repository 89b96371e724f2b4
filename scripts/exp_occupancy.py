#!/usr/bin/env python
"""Occupancy experiment for the lane-per-trace kernel: time config-[2]-like
traces (same generator, capacity scaled with n so that rho stays 2) with n =
64 / 32 / 16 containers under a cap on resident CTAs per SM
(CONVGPU_PER_SM_CAP; a CTA is two warps).  With fewer containers per trace
the shared-memory state per warp shrinks, so the same code can run 1, 2, ...
warps per scheduler; the events/s ratio measures what latency hiding buys.

  python scripts/exp_occupancy.py [--traces 1000000]
"""
import argparse
import dataclasses
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--traces", type=int, default=1_000_000)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--kernel", default="lane")
    a = ap.parse_args()
    import torch

    import paper_conf_cluster_kangjkkk17_b200 as cg
    w2 = W.CONFIGS["c2"]
    res = []
    for n, caps in ((64, (1, 2)), (32, (1, 2, 3, 4)), (16, (2, 4, 6, 8))):
        g = dataclasses.replace(w2.gen, n=n)
        cap = w2.cap * n // 64
        tr = cg.generate(g, 0, a.traces)
        out = cg.alloc_out(a.traces, n)
        for pc in caps:
            os.environ["CONVGPU_PER_SM_CAP"] = str(pc)
            ms = {}
            for pol in W.POLICIES:
                out.stats.zero_()
                cg.replay(tr, cap, pol, out, kernel=a.kernel)
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                best = 1e9
                for _ in range(a.reps):
                    e0.record()
                    cg.replay(tr, cap, pol, out, kernel=a.kernel)
                    e1.record()
                    torch.cuda.synchronize()
                    best = min(best, e0.elapsed_time(e1))
                ms[pol] = round(best, 3)
            ev = a.traces * n * 5
            r = {"n": n, "ctas_per_sm": pc, "warps_per_sm": 2 * pc, "ms": ms,
                 "ev_per_s": {p: ev / (m / 1e3) for p, m in ms.items()}}
            print(json.dumps(r), flush=True)
            res.append(r)
        del tr, out
        torch.cuda.empty_cache()
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    with open(os.path.join(ROOT, "gpurun_out", "exp_occupancy.json"), "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
