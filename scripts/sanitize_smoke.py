"""Small replay of every kernel variant / policy (incl. the literal reading)
for compute-sanitizer runs: memcheck, racecheck, synccheck, initcheck."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
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
print("sanitize smoke done")
