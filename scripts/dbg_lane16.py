"""Debug helper: one small lane16 replay per policy (run under compute-sanitizer)."""
import os
import sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
import workloads as W  # noqa: E402
import paper_conf_cluster_kangjkkk17_b200 as cg  # noqa: E402

w = W.CONFIGS["c2"]
N = int(sys.argv[1]) if len(sys.argv) > 1 else 300
pols = sys.argv[2].split(",") if len(sys.argv) > 2 else list(W.POLICIES)
tr = cg.generate(w.gen, 0, N)
for p in pols:
    out = cg.alloc_out(N, 64)
    cg.replay(tr, w.cap, p, out, kernel="lane16")
    torch.cuda.synchronize()
    print(p, cg.stats_dict(out.stats_np()), flush=True)
