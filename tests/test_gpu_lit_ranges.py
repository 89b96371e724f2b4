"""R1-LIT (NEXT-1) at scale on the compact kernel: 2^20-trace ranges of
config [4] at ρ = 3 and 5 (Random-Fit deadlocks part of them under the
literal reading), all four policies, against the oracle's range digests and
statistics in tests/golden/lit_range_digests.json (written by
scripts/lit_oracle_digests.py from the C oracle only).  Statistics-only
launches through the admission scratch, as the ρ sweep runs them."""
import json
import os

import numpy as np
import pytest

import workloads as W

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden", "lit_range_digests.json")


def _golden():
    if not os.path.exists(GOLDEN):
        pytest.skip("run scripts/lit_oracle_digests.py first")
    with open(GOLDEN) as f:
        return json.load(f)


@pytest.mark.parametrize("rho", [3, 5])
@pytest.mark.parametrize("policy", ["fifo", "best_fit", "recent_fit", "random_fit"])
def test_literal_range_digests(rho, policy):
    import torch

    import paper_conf_cluster_kangjkkk17_b200 as cg
    g = _golden()
    rs, seed = g["range_size"], g["rand_seed"]
    ranges = sorted(int(r) for r in g["rhos"].get(str(rho), {}).get(policy, {}))
    if not ranges:
        pytest.skip("no oracle ranges")
    w = W.rho_sweep(rho, rand_seed=seed)
    nr = max(ranges) + 1
    for r in ranges:
        tr = cg.generate(w.gen, r * rs, rs)
        out = cg.alloc_out(rs, 64, full=False, summary=False, range_count=nr, range_size=rs)
        cg.replay(tr, w.cap, policy + "+literal", out, rand_seed=seed, kernel="lane16")
        torch.cuda.synchronize()
        want = g["rhos"][str(rho)][policy][str(r)]
        rd = out.range_digest.cpu().numpy().view(np.uint64)
        assert "%016x" % int(rd[r]) == want["digest"], (rho, policy, r)
        st = cg.stats_dict(out.stats_np())
        for k in ("traces", "events", "sum_wait", "sum_makespan", "n_select", "flag_count"):
            assert st[k] == want[k], (rho, policy, r, k)
