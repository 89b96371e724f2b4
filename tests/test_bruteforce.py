"""Config [0]: brute-force enumeration on tiny traces (CPU seconds).

oracle/bruteforce.py explores every selection choice (and, with
permute_ties, every order of same-tick events).  It asserts on every path the
paper's guarantees — no deadlock (P:7), memory in use within capacity,
admitted containers keep their declared limit — and for each policy
the single canonical path that obeys the policy's rule must equal
the C oracle's answer field by field.
"""
import time

import pytest

import workloads as W
from oracle import bruteforce as B

KEYS = ["admit_tick", "admit_rank", "wait", "finish", "makespan", "peak_reserved",
        "peak_used", "sum_wait", "n_rejected", "n_select", "flags"]
POLS = ["fifo", "best_fit", "recent_fit", "random_fit"]


def _check_batch(orc, b, cap, ovh, permute, seed=7, max_paths=20000):
    multi = paths_total = 0
    for i in range(b.count):
        tr = dict(arrival=b.arrival[i], limit=b.limit[i], delta=b.delta[i], arg=b.arg[i])
        paths = B.explore(tr, cap, ovh=ovh, tid=i, seed=seed, permute_ties=permute,
                          max_paths=max_paths)
        paths_total += len(paths)
        if any(len(ch[2]) > 1 for _, _, _, chs in paths for ch in chs):
            multi += 1
        for p in POLS:
            r = orc.replay_trace(tr["arrival"], tr["limit"], tr["delta"], tr["arg"], cap, p,
                                 tid=i, seed=seed, ovh=ovh)
            assert r["violation"] == 0
            cand = [o for o, ob, can, _ in paths if p in ob and can]
            assert len(cand) == 1
            for k in KEYS:
                assert cand[0][k] == r[k], (i, p, k, cand[0][k], r[k])
            # every oracle outcome is one of the explored outcomes
            assert any(all(o[k] == r[k] for k in KEYS) for o, _, _, _ in paths)
    return multi, paths_total


def test_fig3_all_interleavings(orc):
    f = W.fig3_fixture()
    paths = B.explore(f, f["cap"], permute_ties=True)
    assert len(paths) > 1
    g = [o for o, ob, can, _ in paths if can]
    assert len(g) == 1 and g[0]["admit_tick"] == [0, 0, 50, 150]


@pytest.mark.parametrize("mode", ["valid", "delayed", "over", "badfree"])
def test_selection_choices_n5(orc, mode):
    t0 = time.time()
    b = W.random_batch(2, 250, 5, 4, 8, mode=mode, max_arrival_step=1,
                       limit_choices=range(1, 9))
    multi, paths = _check_batch(orc, b, 8, 0, permute=False)
    assert multi > 30 or mode == "badfree"
    assert time.time() - t0 < 60


@pytest.mark.parametrize("ovh", [0, 1])
def test_selection_choices_with_overhead(orc, ovh):
    b = W.random_batch(4, 200, 5, 4, 8, ovh=ovh, mode="valid", max_arrival_step=1,
                       limit_choices=range(1, 9))
    _check_batch(orc, b, 8, ovh, permute=False)


def test_same_tick_interleavings_n3(orc):
    b = W.random_batch(2, 250, 3, 3, 8, mode="valid", max_arrival_step=1,
                       limit_choices=range(1, 9))
    _check_batch(orc, b, 8, 0, permute=True)


def test_same_tick_interleavings_n4(orc):
    b = W.random_batch(5, 40, 4, 3, 8, mode="delayed", max_arrival_step=2,
                       limit_choices=range(1, 9))
    _check_batch(orc, b, 8, 0, permute=True, max_paths=50000)


@pytest.mark.parametrize("mode", ["valid", "delayed", "over"])
def test_literal_reading_policy_paths_match_oracle(orc, mode):
    """R1-LIT (NEXT-1): the explorer's literal dispatch (any paused container
    at every release, partial holds kept) contains the oracle's answer for
    each policy as the canonical path obeying that policy's rule; deadlocks
    are outcomes here, not violations."""
    b = W.random_batch(7, 200, 4, 3, 8, mode=mode, max_arrival_step=1,
                       limit_choices=range(1, 9))
    dead = 0
    for i in range(b.count):
        tr = dict(arrival=b.arrival[i], limit=b.limit[i], delta=b.delta[i], arg=b.arg[i])
        paths = B.explore(tr, 8, tid=i, seed=3, lit=True)
        dead += any(o["flags"] & 1 for o, _, _, _ in paths)
        for k, p in enumerate(POLS):
            r = orc.replay_trace(tr["arrival"], tr["limit"], tr["delta"], tr["arg"], 8,
                                 k | 0x100, tid=i, seed=3)
            assert r["violation"] == 0
            cand = [o for o, ob, can, _ in paths if p in ob and can]
            assert len(cand) == 1
            for key in KEYS:
                assert cand[0][key] == r[key], (i, p, key)
    assert dead > 0  # the literal reading admits deadlocking schedules
