"""Small replay of every kernel variant / policy (incl. the literal reading),
the host-memory path and the NEXT-3 wrapper kernel for compute-sanitizer runs: memcheck,
racecheck, synccheck, initcheck."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_cluster_kangjkkk17_b200 as cg  # noqa: E402
import workloads as W  # noqa: E402

for cfg in ("c1", "c2", "mimic"):
    w = W.CONFIGS[cfg]
    N = 700 if cfg == "c2" else 300
    tr = cg.generate(w.gen, 0, N)
    for kernel in ("warp", "lane"):
        for pol in W.POLICIES:
            for name in (pol, pol + "+literal"):
                if kernel == "lane" and name.endswith("literal"):
                    continue
                out = cg.alloc_out(N, w.gen.n, range_count=1, range_size=1 << 20)
                cg.replay(tr, w.cap, name, out, rand_seed=3, ovh=w.ovh, kernel=kernel)
torch.cuda.synchronize()
b = W.random_batch(5, 200, 7, 5, 16, ovh=2, mode="mixed", limit_choices=range(0, 17))
tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg)
for kernel in ("warp", "lane"):
    for pol in W.POLICIES:
        cg.replay(tr, 16, pol, cg.alloc_out(200, 7), ovh=2, kernel=kernel)
torch.cuda.synchronize()
# the compact lane-per-trace kernel (n = 64, K = 4): config [2] (+ rho 8, whose
# limits exceed 16 bits and go through the marked 32-bit fallback launch) and
# a mixed edge-case batch with context overhead
for w in (W.CONFIGS["c2"], W.rho_sweep(8, rand_seed=3)):
    tr = cg.generate(w.gen, 0, 700)
    for pol in W.POLICIES:
        cg.replay(tr, w.cap, pol, cg.alloc_out(700, 64, range_count=1, range_size=1 << 20),
                  rand_seed=3, ovh=w.ovh, kernel="lane16")
b = W.random_batch(6, 300, 64, 4, 64, ovh=1, mode="mixed", limit_choices=range(0, 65))
tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg)
for pol in W.POLICIES:
    cg.replay(tr, 64, pol, cg.alloc_out(300, 64), ovh=1, kernel="lane16")
    # R1-LIT on the compact kernel (+ the warp kernel's marked-only pass) and
    # summary-only launches through the admission scratch (round 2)
    cg.replay(tr, 64, pol + "+literal", cg.alloc_out(300, 64), ovh=1, kernel="lane16")
    cg.replay(tr, 64, pol, cg.alloc_out(300, 64, full=False), ovh=1, kernel="lane16")
# Best-Fit limit classes: <= 8 distinct limits stay on the compact kernel
b8 = W.random_batch(7, 300, 64, 4, 256, mode="valid", limit_choices=[0, 13, 62, 105, 148, 165, 201, 256])
tr8 = cg.traces_from_numpy(b8.arrival, b8.limit, b8.delta, b8.arg)
cg.replay(tr8, 256, "best_fit", cg.alloc_out(300, 64), kernel="lane16")
w4 = W.rho_sweep(8, rand_seed=3)
tr4 = cg.generate(w4.gen, 0, 300)
# the 17-bit layout as the first pass (rho 8) and a batch whose deltas exceed
# 16 bits (marked by the 16-bit and the 17-bit passes, replayed by the 32-bit)
for pol in W.POLICIES:
    cg.replay(tr4, w4.cap, pol, cg.alloc_out(300, 64), rand_seed=3, kernel="lane16w")
    cg.replay(tr4, w4.cap, pol, cg.alloc_out(300, 64, full=False), rand_seed=3, kernel="lane16w")
bd = W.random_batch(8, 300, 64, 4, 200, mode="valid", limit_choices=range(0, 201))
dd = bd.delta.copy()
dd[::3, 1, 0] = 0x10000
trd = cg.traces_from_numpy(bd.arrival, bd.limit, dd, bd.arg)
for pol in W.POLICIES:
    cg.replay(trd, 200, pol, cg.alloc_out(300, 64), kernel="lane16")
for pol in W.POLICIES:
    cg.replay(tr4, w4.cap, pol + "+literal", cg.alloc_out(300, 64), rand_seed=3, kernel="lane16")
torch.cuda.synchronize()
# the 16-bit host format: device packer, host path with the unpack kernel
w2 = W.CONFIGS["c2"]
g2 = cg.generate(w2.gen, 0, 20_000)
t16, oor = cg.pack16(g2)
h16 = t16.pin()
summ16 = np.zeros((4, 20_000), cg.SUMMARY_DTYPE)
cg.replay_host16(h16, w2.cap, W.POLICIES, chunk=9_000, summary=summ16, rand_seed=3)
torch.cuda.synchronize()
# the host-memory path (two copy streams, double-buffered chunks, AUTO kernel)
w = W.CONFIGS["c2"]
g = cg.generate(w.gen, 0, 40_000)
h = [t.cpu() for t in (g.arrival, g.limit, g.op_delta, g.op_arg)]
summ = np.zeros((4, 40_000), cg.SUMMARY_DTYPE)
cg.replay_host(*h, w.cap, W.POLICIES, chunk=19_000, summary=summ, rand_seed=3)
torch.cuda.synchronize()
# NEXT-3 wrapper kernel: the n = 64 / K = 4 fast path, K = 4 and generic shapes
import numpy as np  # noqa: E402
for (N, n, K) in ((300, 64, 4), (97, 5, 4), (50, 7, 8)):
    api = W.random_api_batch(9, N, n, K, "mixed")
    t = torch.from_numpy(np.ascontiguousarray(api).view(np.uint32).reshape(N, K, n, 4)
                         .view(np.int32)).cuda()
    for pitch in (512, 1000, 0):
        cg.wrap_ops(t, n, K, pitch_align=pitch)
torch.cuda.synchronize()
print("sanitize smoke done")
