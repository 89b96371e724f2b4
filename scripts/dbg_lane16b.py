"""Debug: lane16 vs oracle on a few config-[2] traces; dump the first INVALID_FREE."""
import os
import sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402
import workloads as W  # noqa: E402
import oracle  # noqa: E402
import paper_conf_cluster_kangjkkk17_b200 as cg  # noqa: E402

w = W.CONFIGS["c2"]
N = 40
tr = cg.generate(w.gen, 0, N)
out = cg.alloc_out(N, 64)
cg.replay(tr, w.cap, "fifo", out, kernel="lane16")
torch.cuda.synchronize()
s = out.summary_np()
ref = oracle.replay_range(w, "fifo", 0, N, full=True)
D = tr.op_delta.cpu().numpy().view(np.uint32)
R = tr.op_arg.cpu().numpy().view(np.uint32)
L = tr.limit.cpu().numpy().view(np.uint32)
for i in range(N):
    if s["flags"][i] & 8:
        d0 = int(s["makespan"][i]); c, k, pc = d0 & 255, (d0 >> 8) & 255, d0 >> 16
        print("trace", i, "c", c, "k", k, "pre_c", pc, "r", int(s["peak_reserved"][i]), "used", int(s["peak_used"][i]),
              "ust %08x" % int(s["n_rejected"][i]), "sd %08x" % int(s["n_select"][i]), "events", int(s["sum_wait"][i]))
        print("  L", L[i, c], "ops", [(int(R[i, kk, c]) >> 30, int(R[i, kk, c]) & 0x3FFFFFFF, int(D[i, kk, c])) for kk in range(4)])
        print("  oracle admit", ref["admit_tick"][i][c], "wait", ref["wait"][i][c], "finish", ref["finish"][i][c])
        break
print("flags", [int(x) for x in s["flags"]])
