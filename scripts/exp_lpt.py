#!/usr/bin/env python
"""Kernel-tuning sweep: time the replay kernel per policy on config [2] for
each value of an environment knob read by libconvgpu at launch, and check the
statistics record (digest sum, events, ...) is unchanged across values.

  python scripts/exp_lpt.py --env CONVGPU_LPT_DTHRESH --values 0,4,8,16 [--kernel lane]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--env", default="CONVGPU_LPT_DTHRESH")
    ap.add_argument("--values", default="0")
    ap.add_argument("--kernel", default="lane")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--traces", type=int, default=0)
    a = ap.parse_args()
    import torch

    import paper_conf_cluster_kangjkkk17_b200 as cg
    w = W.CONFIGS["c2"]
    count = a.traces or w.n_traces
    tr = cg.generate(w.gen, 0, count)
    out = cg.alloc_out(count, w.gen.n)
    ref = {}
    for v in a.values.split(","):
        os.environ[a.env] = v
        ms, tot_ev = {}, 0
        for pol in W.POLICIES:
            out.stats.zero_()
            cg.replay(tr, w.cap, pol, out, rand_seed=w.rand_seed, ovh=w.ovh, kernel=a.kernel)
            torch.cuda.synchronize()
            st = cg.stats_dict(out.stats_np())
            if pol in ref:
                assert st == ref[pol], (v, pol)
            ref[pol] = st
            tot_ev += st["events"]
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            best = 1e9
            for _ in range(a.reps):
                e0.record(); cg.replay(tr, w.cap, pol, out, rand_seed=w.rand_seed, ovh=w.ovh,
                                       kernel=a.kernel); e1.record()
                torch.cuda.synchronize()
                best = min(best, e0.elapsed_time(e1))
            ms[pol] = round(best, 2)
        dig = ",".join("%04x" % (ref[p]["digest_sum"] >> 48) for p in W.POLICIES)
        print(f"{a.env}={v} {a.kernel} {tot_ev / (sum(ms.values()) / 1e3):.3e} ev/s {ms} dig={dig}",
              flush=True)


if __name__ == "__main__":
    main()
