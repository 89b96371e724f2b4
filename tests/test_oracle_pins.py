"""Pins of the C oracle to things other than itself (paper values, closed
forms, published constants, invariants).  CPU only."""
import numpy as np
import pytest

import workloads as W
from conftest import golden
from workloads import ALLOC, FINISH, FREE, NOP, op

KEYS = ["admit_tick", "admit_rank", "wait", "finish", "makespan", "peak_reserved",
        "peak_used", "sum_wait", "n_rejected", "n_select", "flags"]
POLS = ["fifo", "best_fit", "recent_fit", "random_fit"]


def h(x):
    return int(x, 16)


# --- published constants -------------------------------------------------
def test_philox_kat(orc):
    from oracle import bruteforce
    for v in golden("philox_kat.json")["vectors"]:
        ctr = [h(x) for x in v["ctr"]]
        key = [h(x) for x in v["key"]]
        out = [h(x) for x in v["out"]]
        assert orc.philox4x32_10(ctr, key) == out
        assert bruteforce.philox4x32_10(ctr, key) == out


def test_splitmix64_published_outputs(orc):
    g = golden("splitmix64.json")
    gamma = h(g["gamma"])
    for k, want in enumerate(g["outputs_seed0"], start=1):
        assert orc.mix64((k * gamma) % 2**64) == h(want)


# --- the paper's worked example (Fig. 3) -----------------------
@pytest.mark.parametrize("policy", POLS)
def test_fig3_narrative(orc, policy):
    g = golden("fig3.json")["expected_all_policies"]
    f = W.fig3_fixture()
    r = orc.replay_trace(f["arrival"], f["limit"], f["delta"], f["arg"], f["cap"], policy)
    for k in KEYS + ["events"]:
        assert r[k] == g[k], k
    assert r["violation"] == 0


def test_fig3_digest_definition(orc):
    """The digest is the DESIGN.md R20 sum; recompute it from the outputs."""
    f = W.fig3_fixture()
    r = orc.replay_trace(f["arrival"], f["limit"], f["delta"], f["arg"], f["cap"], "fifo")
    M = 2**64
    d = 0
    for c in range(4):
        h1 = orc.mix64((c << 56) ^ (r["admit_rank"][c] << 48) ^ r["admit_tick"][c])
        d += orc.mix64(h1 ^ ((r["wait"][c] << 32) | r["finish"][c]))
    d += orc.mix64((r["makespan"] << 32) | r["peak_reserved"])
    d += orc.mix64((r["peak_used"] << 32) | r["flags"])
    d += orc.mix64(r["sum_wait"])
    d += orc.mix64((r["n_rejected"] << 32) | r["n_select"])
    assert r["digest"] == d % M


# --- closed forms ----------------------------------------------------------
def _single_alloc_trace(arrival, limit, dur):
    n = len(arrival)
    delta = np.zeros((2, n), np.uint32)
    arg = np.zeros((2, n), np.uint32)
    for c in range(n):
        arg[0, c] = op(ALLOC, limit[c])
        arg[1, c] = op(FINISH)
        delta[1, c] = dur[c]
    return np.array(arrival, np.uint32), np.array(limit, np.uint32), delta, arg


def test_fifo_reduces_to_lindley_fcfs(orc):
    """Every L_i > cap/2 and programs [ALLOC L_i @0, FINISH @d_i]: only one
    container can hold memory, so FIFO is an FCFS single server:
    finish_i = max(arrival_i, finish_{i-1}) + d_i, wait_i = start_i - arrival_i."""
    rng = np.random.default_rng(11)
    cap = 1000
    for _ in range(400):
        n = int(rng.integers(1, 65))
        arrival = np.cumsum(rng.integers(0, 40, n)).tolist()
        limit = rng.integers(cap // 2 + 1, cap + 1, n).tolist()
        dur = rng.integers(0, 60, n).tolist()
        a, L, d, g = _single_alloc_trace(arrival, limit, dur)
        r = orc.replay_trace(a, L, d, g, cap, "fifo")
        prev = 0
        for i in range(n):
            start = max(arrival[i], prev)
            prev = start + dur[i]
            assert r["finish"][i] == prev
            assert r["wait"][i] == start - arrival[i]
            assert r["admit_tick"][i] == start
            assert r["admit_rank"][i] == i
        assert r["makespan"] == prev - arrival[0]
        assert r["flags"] == 0 and r["violation"] == 0


@pytest.mark.parametrize("policy", POLS)
def test_no_contention(orc, policy):
    """sum L <= cap: nobody is ever paused; admit at arrival; finish =
    arrival + sum of deltas; no selection happens (P:139 needs insufficiency)."""
    b = W.random_batch(5, 200, 6, 4, 60, mode="valid", limit_choices=range(0, 11))
    for i in range(b.count):
        r = orc.replay_trace(b.arrival[i], b.limit[i], b.delta[i], b.arg[i], 60, policy)
        assert r["n_select"] == 0 and r["sum_wait"] == 0
        for c in range(6):
            assert r["admit_tick"][c] == b.arrival[i][c]
            assert r["finish"][c] == int(b.arrival[i][c]) + int(b.delta[i][:, c].sum())
        assert sorted(r["admit_rank"]) == list(range(6))
        assert r["peak_reserved"] <= int(b.limit[i].sum())


def test_best_fit_equals_fifo_for_equal_limits(orc):
    """Equal limits and single-ALLOC programs: every paused container has the
    same shortfall L, so Best-Fit's tie-break (lowest index) is FIFO's rule."""
    rng = np.random.default_rng(3)
    for _ in range(300):
        n = int(rng.integers(2, 40))
        cap = 1000
        L = int(rng.integers(1, cap + 1))
        arrival = np.cumsum(rng.integers(0, 5, n)).tolist()
        dur = rng.integers(0, 50, n).tolist()
        a, Lm, d, g = _single_alloc_trace(arrival, [L] * n, dur)
        rf = orc.replay_trace(a, Lm, d, g, cap, "fifo")
        rb = orc.replay_trace(a, Lm, d, g, cap, "best_fit")
        for k in KEYS:
            assert rf[k] == rb[k], k


def test_single_candidate_all_policies_identical(orc):
    """When every selection sees one paused container, the four rules agree."""
    b = W.random_batch(9, 400, 4, 3, 8, mode="valid", limit_choices=range(1, 9))
    agree = 0
    for i in range(b.count):
        rs = [orc.replay_trace(b.arrival[i], b.limit[i], b.delta[i], b.arg[i], 8, p)
              for p in POLS]
        if rs[0]["n_select"] == 0:
            for r in rs[1:]:
                assert all(r[k] == rs[0][k] for k in KEYS)
                agree += 1
    assert agree > 100


# --- specific semantics ------------------------------------------------------
def test_context_overhead_first_alloc(orc):
    """66 MiB are charged at a pid's first allocation."""
    a = np.array([0], np.uint32)
    L = np.array([100], np.uint32)
    delta = np.zeros((4, 1), np.uint32)
    arg = np.array([[op(ALLOC, 34)], [op(ALLOC, 1)], [op(FREE, 34)], [op(FINISH)]], np.uint32)
    r = orc.replay_trace(a, L, delta, arg, 200, "fifo", ovh=66)
    assert r["n_rejected"] == 1 and r["peak_used"] == 100 and r["flags"] == 0
    r0 = orc.replay_trace(a, L, delta, arg, 200, "fifo", ovh=0)
    assert r0["n_rejected"] == 0 and r0["peak_used"] == 35


def test_reject_over_limit_continues(orc):
    """an allocation over the declared limit is denied; the
    program keeps running (R10)."""
    a = np.array([0, 0], np.uint32)
    L = np.array([10, 10], np.uint32)
    delta = np.array([[0, 0], [5, 5], [5, 5]], np.uint32)
    arg = np.array([[op(ALLOC, 11), op(ALLOC, 10)], [op(ALLOC, 10), op(NOP)],
                    [op(FINISH), op(FINISH)]], np.uint32)
    r = orc.replay_trace(a, L, delta, arg, 20, "fifo")
    assert r["n_rejected"] == 1 and r["finish"] == [10, 10] and r["peak_used"] == 20


def test_free_keeps_assignment(orc):
    """R11: cudaFree lowers usage only; memory returns to others at FINISH."""
    a = np.array([0, 1], np.uint32)
    L = np.array([10, 10], np.uint32)
    delta = np.array([[0, 0], [1, 0], [100, 0]], np.uint32)
    arg = np.array([[op(ALLOC, 10), op(ALLOC, 10)], [op(FREE, 10), op(NOP)],
                    [op(FINISH), op(FINISH)]], np.uint32)
    r = orc.replay_trace(a, L, delta, arg, 10, "fifo")
    # container 1 waits for container 0's exit at t=101, not its free at t=1
    assert r["admit_tick"] == [0, 101] and r["wait"] == [0, 100]


def _flags_only(r, n):
    assert r["admit_tick"] == [0xFFFFFFFF] * n and r["admit_rank"] == [0xFF] * n
    assert r["wait"] == [0] * n and r["finish"] == [0] * n
    assert r["makespan"] == 0 and r["peak_reserved"] == 0 and r["n_select"] == 0


def test_static_flags(orc):
    f = W.fig3_fixture()
    base = {k: np.array(f[k]).copy() for k in ("arrival", "limit", "delta", "arg")}
    # INVALID_LIMIT (R15)
    x = {k: v.copy() for k, v in base.items()}
    x["limit"][2] = 8193
    r = orc.replay_trace(x["arrival"], x["limit"], x["delta"], x["arg"], 8192, "fifo")
    assert r["flags"] == 1 << 2 and r["events"] == 0
    _flags_only(r, 4)
    # UNSORTED_ARRIVAL
    x = {k: v.copy() for k, v in base.items()}
    x["arrival"][3] = 5
    r = orc.replay_trace(x["arrival"], x["limit"], x["delta"], x["arg"], 8192, "fifo")
    assert r["flags"] == 1 << 4
    _flags_only(r, 4)
    # BAD_PROGRAM: FINISH not last / last not FINISH
    x = {k: v.copy() for k, v in base.items()}
    x["arg"][1, 0] = op(FINISH)
    r = orc.replay_trace(x["arrival"], x["limit"], x["delta"], x["arg"], 8192, "fifo")
    assert r["flags"] == 1 << 6
    x = {k: v.copy() for k, v in base.items()}
    x["arg"][2, 3] = op(NOP)
    r = orc.replay_trace(x["arrival"], x["limit"], x["delta"], x["arg"], 8192, "fifo")
    assert r["flags"] == 1 << 6
    # TICK_RANGE (R19): horizon max arrival + sum deltas >= 2^26
    x = {k: v.copy() for k, v in base.items()}
    # fig3: max arrival 20, other deltas sum 260 -> horizon = 280 + X
    x["delta"][2, 0] = (1 << 26) - 280
    r = orc.replay_trace(x["arrival"], x["limit"], x["delta"], x["arg"], 8192, "fifo")
    assert r["flags"] == 1 << 5
    x["delta"][2, 0] = (1 << 26) - 281   # horizon 2^26 - 1: representable
    r = orc.replay_trace(x["arrival"], x["limit"], x["delta"], x["arg"], 8192, "fifo")
    assert r["flags"] == 0
    # several static flags at once accumulate
    x = {k: v.copy() for k, v in base.items()}
    x["limit"][0] = 9000
    x["arrival"][1] = 30
    r = orc.replay_trace(x["arrival"], x["limit"], x["delta"], x["arg"], 8192, "fifo")
    assert r["flags"] == (1 << 2) | (1 << 4)


def test_invalid_free_stops(orc):
    a = np.array([0], np.uint32)
    L = np.array([10], np.uint32)
    delta = np.zeros((3, 1), np.uint32)
    arg = np.array([[op(ALLOC, 4)], [op(FREE, 5)], [op(FINISH)]], np.uint32)
    r = orc.replay_trace(a, L, delta, arg, 10, "fifo")
    assert r["flags"] == 1 << 3 and r["events"] == 3
    _flags_only(r, 1)


def test_finish_releases_unfreed_memory(orc):
    """P:110/P:137 (R18): exit drops every allocation of the pid."""
    a = np.array([0, 0], np.uint32)
    L = np.array([8, 8], np.uint32)
    delta = np.array([[0, 0], [7, 0]], np.uint32)
    arg = np.array([[op(ALLOC, 8), op(ALLOC, 8)], [op(FINISH), op(FINISH)]], np.uint32)
    r = orc.replay_trace(a, L, delta, arg, 8, "fifo")
    assert r["admit_tick"] == [0, 7] and r["finish"] == [7, 7]


def test_random_fit_is_uniform(orc):
    """P:145 'selects randomly among paused containers': chi-square over
    seeds on a selection with m = 3 candidates (statistical, not parity)."""
    n = 5
    arrival = np.array([0, 1, 2, 3, 4], np.uint32)
    limit = np.array([4] * n, np.uint32)
    delta = np.zeros((2, n), np.uint32)
    delta[1, :] = 10
    arg = np.array([[op(ALLOC, 4)] * n, [op(FINISH)] * n], np.uint32)
    counts = np.zeros(n, int)
    S = 3000
    for seed in range(S):
        r = orc.replay_trace(arrival, limit, delta, arg, 4, "random_fit", seed=seed)
        counts[r["admit_rank"].index(2)] += 1
    assert counts[0] == 0 and counts[1] == 0
    exp = S / 3
    chi2 = float(((counts[2:] - exp) ** 2 / exp).sum())
    assert chi2 < 13.8  # p = 0.001 at 2 dof


# --- invariants on the configs --------------------------------------------
@pytest.mark.parametrize("cfg", ["c1", "c2", "mimic"])
@pytest.mark.parametrize("policy", POLS)
def test_invariants_on_configs(orc, cfg, policy):
    """Per-event invariants + no deadlock (P:7) +
    FIFO admits in arrival order when first ALLOCs are immediate."""
    w = W.CONFIGS[cfg]
    r = orc.replay_range(w, policy, 0, 150, full=True, check=True)
    assert r["rc"] == 0
    st = r["stats"]
    assert st["flag_count"] == [0] * 8
    assert st["events"] == 150 * w.events_per_trace()
    assert (r["peak_reserved"] <= w.cap).all()
    assert (r["peak_used"] <= r["peak_reserved"]).all()
    if policy == "fifo":
        for i in range(150):
            ranks = r["admit_rank"][i]
            adm = ranks[ranks != 0xFF]
            assert (np.diff(adm.astype(int)) > 0).all()


@pytest.mark.parametrize("mode", ["valid", "delayed", "over", "badfree", "mixed"])
@pytest.mark.parametrize("policy", POLS)
def test_invariants_on_edge_batches(orc, mode, policy):
    b = W.random_batch(21, 300, 7, 5, 16, ovh=2, mode=mode, limit_choices=range(0, 17))
    r = orc.replay_batch(b, 16, policy, ovh=2, check=True)
    assert r["rc"] == 0
    assert r["stats"]["flag_count"][0] == 0 and r["stats"]["flag_count"][1] == 0


def test_generator_recipe(orc):
    """Input recipe: classes uniform over the table (P:179
    'randomly'), L = class*num/den, arrival = c*iat, program sums."""
    from oracle import bruteforce
    w = W.CONFIGS["c2"]
    g = w.gen
    counts = np.zeros(6, int)
    for tid in range(400):
        a, L, d, arg = orc.generate(g, tid)
        assert (a == np.arange(64) * g.iat).all()
        for c in range(64):
            x = bruteforce.philox4x32_10([tid, 0, c, 0], [g.gen_seed & 0xFFFFFFFF, g.gen_seed >> 32])
            k = (x[0] * 6) >> 32
            counts[k] += 1
            assert L[c] == g.class_mib[k] * g.num // g.den
            dur = g.dur_base + g.dur_step * k
            assert int(d[:, c].sum()) == dur
            sizes = arg[:, c] & 0x3FFFFFFF
            kinds = arg[:, c] >> 30
            assert list(kinds) == [ALLOC, ALLOC, FREE, FINISH]
            assert sizes[0] + sizes[1] == L[c] and sizes[2] == sizes[0]
    exp = counts.sum() / 6
    assert float(((counts - exp) ** 2 / exp).sum()) < 20.5  # p=0.001, 5 dof


# --- NEXT-1: the literal re-select-on-every-release reading (R1-LIT) -------
LIT = 0x100


def _survey_counterexample():
    """cap 20; G (L 10) and F (L 4) run from t=0, G
    exits at t=2, F at t=100; X (L 20) arrives at t=1 and Z (L 18) at t=3,
    both ALLOC their whole limit at t=50 and run 10 more ticks."""
    arrival = np.array([0, 0, 1, 3], np.uint32)
    limit = np.array([10, 4, 20, 18], np.uint32)
    delta = np.array([[0, 0, 49, 47], [2, 100, 10, 10]], np.uint32)
    arg = np.array([[op(ALLOC, 10), op(ALLOC, 4), op(ALLOC, 20), op(ALLOC, 18)],
                    [op(FINISH)] * 4], np.uint32)
    return arrival, limit, delta, arg


@pytest.mark.parametrize("policy", POLS)
def test_literal_reading_deadlocks_where_sticky_does_not(orc, policy):
    """P:7 claims the policies prevent deadlock.  Under R1 (sticky target) the
    counterexample completes; under the literal reading every policy leaves X
    and Z paused on partial holds that can never be completed."""
    a, L, d, g = _survey_counterexample()
    r = orc.replay_trace(a, L, d, g, 20, policy)
    assert r["flags"] == 0 and r["finish"][2] > 0 and r["finish"][3] > 0
    rl = orc.replay_trace(a, L, d, g, 20, POLS.index(policy) | LIT)
    assert rl["flags"] == 1 and rl["violation"] == 0  # DEADLOCK, ledger intact


def test_literal_reading_contradicts_fig3_for_best_fit(orc):
    """Under the literal reading Best-Fit gives B's 3072 MiB to D (the closest
    fit) at t=50, not to C as Fig. 3d narrates — one reason DESIGN.md
    takes the sticky reading R1."""
    f = W.fig3_fixture()
    r = orc.replay_trace(f["arrival"], f["limit"], f["delta"], f["arg"], f["cap"], 1 | LIT)
    assert r["admit_tick"][3] == 50 and r["admit_tick"][2] != 50
    r = orc.replay_trace(f["arrival"], f["limit"], f["delta"], f["arg"], f["cap"], 0 | LIT)
    assert r["admit_tick"] == [0, 0, 50, 150]  # FIFO happens to agree


@pytest.mark.parametrize("policy", POLS)
def test_literal_reading_invariants_and_deadlock_rate(orc, policy):
    """The ledger invariants still hold under the literal reading; on the
    paper-mimic workload (one container every 5 s) it deadlocks a
    share of traces that the sticky reading completes."""
    w = W.CONFIGS["mimic"]
    sticky = orc.replay_range(w, policy, 0, 200, check=True)
    lit = orc.replay_range(w, POLS.index(policy) | LIT, 0, 200, check=True)
    assert sticky["rc"] == 0 and lit["rc"] == 0
    assert sticky["stats"]["flag_count"][0] == 0
    assert lit["stats"]["flag_count"][1] == 0  # never overcommits


@pytest.mark.parametrize("case", range(4))
def test_generator_exact_values(orc, case):
    """orc_generate against values derived BY HAND from the recipe
    (tests/golden/generator_cases.json 'work'): the per-op split s1 = e/2,
    s2 = e - s1, d1 = dur/4, d2 = dur/2, d3 = dur - d1 - d2, e = max(L - ovh, 0),
    the jitter term, the class offset, 64-bit trace ids and the K = 2
    program.  Swapping d1/d2 or s1/s2, dropping ovh or the jitter each fail
    one of the four cases."""
    from oracle import bruteforce
    cs = golden("generator_cases.json")["cases"][case]
    g = W.GenParams(**{k: (tuple(v) if k == "class_mib" else v) for k, v in cs["gen"].items()})
    tid, c = cs["tid"], cs["c"]
    # the two Philox words the derivation starts from (Philox is KAT-pinned)
    x = bruteforce.philox4x32_10([tid & 0xFFFFFFFF, tid >> 32, c, 0],
                                 [g.gen_seed & 0xFFFFFFFF, g.gen_seed >> 32])
    assert x[0] == h(cs["x0"]) and x[1] == h(cs["x1"])
    a, L, d, arg = orc.generate(g, tid)
    assert int(a[c]) == cs["arrival"]
    assert int(L[c]) == cs["limit"]
    assert [int(v) for v in d[:, c]] == cs["delta"]
    assert [int(v) >> 30 for v in arg[:, c]] == cs["kind"]
    assert [int(v) & 0x3FFFFFFF for v in arg[:, c]] == cs["size"]
