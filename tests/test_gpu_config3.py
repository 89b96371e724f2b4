"""BASELINE config [3] at full scale: 10^8 traces x 64 containers (config [2]
generator), every policy, compared with the oracle range by range.

The expected per-2^20-trace digests (sum of trace digests mod 2^64, plus
event / wait / makespan / selection totals) are written by
scripts/c3_oracle_digests.py, which runs only the C oracle; this test
regenerates each range on the GPU, replays it in the bench launch
configuration (no per-container outputs, statistics + range digests) and
requires bit-exact agreement on every range the golden file holds."""
import json
import os

import numpy as np
import pytest

import workloads as W

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden", "c3_range_digests.json")
CHUNK_RANGES = 4


def _golden():
    if not os.path.exists(GOLDEN):
        pytest.skip("run scripts/c3_oracle_digests.py first")
    with open(GOLDEN) as f:
        return json.load(f)


@pytest.mark.parametrize("policy", ["fifo", "best_fit", "recent_fit", "random_fit"])
@pytest.mark.parametrize("kernel", ["lane16", "lane"])
def test_config3_range_digests(policy, kernel):
    """kernel: "lane16" = the compact kernel bench.py times (summary-only
    through the admission scratch, as AUTO picks it), "lane" = the 32-bit
    lane kernel."""
    import torch

    import paper_conf_cluster_kangjkkk17_b200 as cg
    g = _golden()
    ranges = sorted(int(r) for r in g["policies"].get(policy, {}))
    if not ranges:
        pytest.skip(f"no oracle ranges for {policy} yet")
    w = W.CONFIGS["c3"]
    rs = g["range_size"]
    assert rs == 1 << 20 and g["n_traces"] == w.n_traces
    nr = (w.n_traces + rs - 1) // rs
    buf = None
    checked = 0
    for c0 in range(0, nr, CHUNK_RANGES):
        want = [r for r in range(c0, min(c0 + CHUNK_RANGES, nr)) if r in ranges]
        if not want:
            continue
        lo, hi = c0 * rs, min((c0 + CHUNK_RANGES) * rs, w.n_traces)
        if buf is None or buf.count < hi - lo:
            buf = cg.empty_traces(CHUNK_RANGES * rs, w.gen.n, w.gen.K)
        tr = cg.Traces(buf.arrival[:hi - lo], buf.limit[:hi - lo], buf.op_delta[:hi - lo],
                       buf.op_arg[:hi - lo])
        cg.generate(w.gen, lo, hi - lo, out=tr)
        out = cg.alloc_out(hi - lo, w.gen.n, full=False, summary=False, range_count=nr,
                           range_size=rs, scratch=kernel == "lane16")
        cg.replay(tr, w.cap, policy, out, rand_seed=w.rand_seed,
                  kernel="auto" if kernel == "lane16" else kernel)
        torch.cuda.synchronize()
        rd = out.range_digest.cpu().numpy().view(np.uint64)
        st = cg.stats_dict(out.stats_np())
        tot_ev = 0
        for r in want:
            assert "%016x" % int(rd[r]) == g["policies"][policy][str(r)]["digest"], (policy, r)
            tot_ev += g["policies"][policy][str(r)]["events"]
            checked += 1
        if len(want) == hi // rs - c0 or hi == w.n_traces:
            exp = [g["policies"][policy].get(str(r)) for r in range(c0, (hi + rs - 1) // rs)]
            if all(e is not None for e in exp):
                assert st["events"] == sum(e["events"] for e in exp)
                assert st["sum_wait"] == sum(e["sum_wait"] for e in exp)
                assert st["n_select"] == sum(e["n_select"] for e in exp)
                assert st["flag_count"] == [0] * 8
    assert checked == len(ranges)
