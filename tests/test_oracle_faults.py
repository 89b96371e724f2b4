"""The oracle's invariant checker is shown to FIRE.

A checker that always returned 0 would pass every "no violation" test in
test_oracle_pins.py.  Here the oracle is rebuilt with one deliberate bug at a
time (-DORC_FAULT=<n>, oracle/oracle.c; the normal build plants none) and each
planted bug must be reported by the per-event invariant checker (violation
codes of check_invariants) or by the per-trace R17 check (code 12), while the
unfaulted build reports nothing on the same traces.  CPU only."""
import pytest

import workloads as W

# fault -> (what it breaks, violation codes that may report it)
FAULTS = {
    1: ("FINISH does not return the assignment to the pool (P:139)", {1}),
    2: ("a fill ignores the target's remaining shortfall, so a > L (P:141)", {3}),
    3: ("an ALLOC is granted beyond the assigned memory (P:78, P:139)", {2}),
    4: ("a resume does not add the suspended time (R17)", {12}),
    5: ("FINISH of the fill target leaves it as target (R20)", {4, 10, 11}),
    6: ("a partially assigned newcomer is admitted (P:141 'until ... reaches')", {5, 6}),
}


@pytest.fixture(scope="module")
def fault_libs(tmp_path_factory, orc):
    d = str(tmp_path_factory.mktemp("orc_fault"))
    return {f: orc.load(orc.build_fault(f, d)) for f in FAULTS}


@pytest.mark.parametrize("fault", sorted(FAULTS))
@pytest.mark.parametrize("policy", ["fifo", "best_fit", "recent_fit", "random_fit"])
def test_checker_fires_on_planted_fault(orc, fault_libs, fault, policy):
    # config [1] traces and small seeded edge-case traces (workloads.random_batch)
    w = W.CONFIGS["c1"]
    b = W.random_batch(5, 400, 5, 4, 16, ovh=1, mode="valid", limit_choices=range(0, 17))
    assert orc.replay_range(w, policy, 0, 40, check=True)["rc"] == 0
    assert orc.replay_batch(b, 16, policy, ovh=1, check=True)["rc"] == 0
    codes = set()
    for r in (orc.replay_range(w, policy, 0, 40, check=True, L=fault_libs[fault]),
              orc.replay_batch(b, 16, policy, ovh=1, check=True, L=fault_libs[fault])):
        if r["rc"] > 1000:
            codes.add(r["rc"] - 1000)
    assert codes, f"fault {fault} ({FAULTS[fault][0]}) went unnoticed"
    assert codes <= FAULTS[fault][1], (fault, codes)


def test_unfaulted_build_is_the_default(orc):
    """build_fault(0) plants nothing: identical results to lib()."""
    import tempfile
    with tempfile.TemporaryDirectory() as d:
        L0 = orc.load(orc.build_fault(0, d))
        w = W.CONFIGS["c2"]
        for policy in ("fifo", "best_fit"):
            a = orc.replay_range(w, policy, 0, 20, check=True)
            b = orc.replay_range(w, policy, 0, 20, check=True, L=L0)
            assert a["rc"] == b["rc"] == 0
            assert (a["digest"] == b["digest"]).all()
