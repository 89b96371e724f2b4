"""Micro-step counters of a LPT16_COUNT build (experiment only): per trace
events / dispatch steps / hazard idles / warp iterations, per policy."""
import os, sys
import numpy as np
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch, workloads as W, paper_conf_cluster_kangjkkk17_b200 as cg
w = W.CONFIGS['c2']; N = 65536; tr = cg.generate(w.gen, 0, N)
for pol in W.POLICIES:
    out = cg.alloc_out(N, w.gen.n)
    cg.replay(tr, w.cap, pol, out, rand_seed=w.rand_seed, ovh=w.ovh, kernel='lane16')
    torch.cuda.synchronize()
    s = out.summary_np()
    ev, ds, hz, it = (s[f].astype(np.float64) for f in ("makespan", "peak_reserved", "peak_used", "n_rejected"))
    wmax = it.reshape(-1, 32).max(1)
    print(pol, "event-steps %.1f dispatch %.1f hazard-idle %.1f lane-iters %.1f warp-iters(max/32) %.1f" % (ev.mean(), ds.mean(), hz.mean(), it.mean(), wmax.mean()))
