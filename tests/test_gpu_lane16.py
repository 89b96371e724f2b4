"""GPU parity of the compact lane-per-trace kernel (csrc/replay_lpt16.cu,
CONVGPU_KERNEL_LANE_COMPACT) against the C oracle, element by element, on
every integer output: configs [2] and [4] (rho 8 has limits above the 16-bit
fields, so its traces go through the marked 17-bit second launch), edge-case
batches with tiny deltas (consecutive events of one container hit the
register-fetch slow path), extreme values (fallback and static flags), a
batch mixing eligible and ineligible traces, and the full-size config [2]
sampled.  Needs a B200: run via gpurun."""
import numpy as np
import pytest

import workloads as W
from test_gpu_parity import POLS, _compare, _compare_stats, _extreme_batch, _gpu_replay

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cg():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_cluster_kangjkkk17_b200 as m
    from paper_conf_cluster_kangjkkk17_b200 import build
    build.build()
    return m


@pytest.mark.parametrize("policy", POLS)
def test_lane16_config2_window_ragged(cg, orc, policy):
    w = W.CONFIGS["c2"]
    base, N = 987_654_321_001, 4_741
    ref = orc.replay_range(w, policy, base, base + N, full=True)
    tr = cg.generate(w.gen, base, N)
    out = _gpu_replay(cg, tr, w.cap, policy, seed=w.rand_seed, kernel="lane16")
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])


@pytest.mark.parametrize("policy", POLS)
@pytest.mark.parametrize("rho", [1, 4, 7, 8])
def test_lane16_rho_sweep(cg, orc, policy, rho):
    w = W.rho_sweep(rho, rand_seed=rho * 7 + 1)
    ref = orc.replay_range(w, policy, 10_000, 11_500, full=True)
    tr = cg.generate(w.gen, 10_000, 1_500)
    for kernel in ("lane16", "lane16w"):
        out = _gpu_replay(cg, tr, w.cap, policy, seed=w.rand_seed, kernel=kernel)
        _compare(cg, out, ref)
        _compare_stats(cg, out, ref["stats"])


EDGE64 = [  # (cap, ovh, mode, count)
    (256, 0, "valid", 700),
    (512, 66, "valid", 500),
    (300, 5, "mixed", 900),
    (128, 0, "over", 500),
    (200, 1, "delayed", 500),
    (256, 0, "badfree", 400),
]


@pytest.mark.parametrize("case", EDGE64, ids=lambda c: f"{c[2]}{c[0]}o{c[1]}")
@pytest.mark.parametrize("policy", POLS)
def test_lane16_edge_batches(cg, orc, policy, case):
    cap, ovh, mode, count = case
    b = W.random_batch(4242 + cap, count, 64, 4, cap, ovh=ovh, mode=mode,
                       limit_choices=range(0, cap + 1))
    base = 7_000_000_000 + cap
    ref = orc.replay_batch(b, cap, policy, tid_base=base, rand_seed=5 + cap, ovh=ovh)
    tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg, trace_id_base=base)
    out = _gpu_replay(cg, tr, cap, policy, seed=5 + cap, ovh=ovh, kernel="lane16")
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])


@pytest.mark.parametrize("policy", POLS)
def test_lane16_extreme_values_and_mixed_batch(cg, orc, policy):
    """Values at the ABI limits (all ineligible or statically flagged),
    interleaved with config-[2] traces that the compact kernel replays."""
    xb, cap, ovh = _extreme_batch(95, 300, 64, 4)
    ref = orc.replay_batch(xb, cap, policy, tid_base=2**63 + 5, rand_seed=2**64 - 1, ovh=ovh)
    tr = cg.traces_from_numpy(xb.arrival, xb.limit, xb.delta, xb.arg, trace_id_base=2**63 + 5)
    out = _gpu_replay(cg, tr, cap, policy, seed=2**64 - 1, ovh=ovh, kernel="lane16")
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])
    # a mixed batch: small-valued traces (compact) next to large-valued ones (fallback)
    sb = W.random_batch(96, 300, 64, 4, 16, ovh=1, mode="mixed", limit_choices=range(0, 17))
    mix = W.Batch(64, 4, *(np.concatenate([getattr(sb, f), getattr(xb, f)])[np.argsort(
        np.arange(600) % 7, kind="stable")] for f in ("arrival", "limit", "delta", "arg")))
    ref = orc.replay_batch(mix, cap, policy, tid_base=11, rand_seed=3, ovh=ovh)
    tr = cg.traces_from_numpy(mix.arrival, mix.limit, mix.delta, mix.arg, trace_id_base=11)
    out = _gpu_replay(cg, tr, cap, policy, seed=3, ovh=ovh, kernel="lane16")
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])


@pytest.mark.parametrize("policy", POLS)
def test_lane16_full_size_sampled(cg, orc, policy):
    """Config [2] at full size in the bench launch configuration (AUTO with full
    outputs = the compact kernel): sampled traces against the oracle one by
    one, stats and range digest against the outputs."""
    w = W.CONFIGS["c2"]
    N = w.n_traces
    tr = cg.generate(w.gen, 0, N)
    rs = 1 << 16
    out = _gpu_replay(cg, tr, w.cap, policy, seed=w.rand_seed, range_size=rs,
                      range_count=(N + rs - 1) // rs)
    s = out.summary_np()
    full = out.full_np()
    rng = np.random.default_rng(11)
    idx = np.unique(np.concatenate([rng.integers(0, N, 200), [0, 1, N - 2, N - 1]]))
    for i in idx:
        ref = orc.replay_range(w, policy, int(i), int(i) + 1, full=True)
        for f in ("makespan", "peak_reserved", "peak_used", "flags", "sum_wait", "n_rejected",
                  "n_select", "digest"):
            assert int(s[f][i]) == int(ref[f][0]), (i, f)
        for f in ("admit_tick", "admit_rank", "wait", "finish"):
            np.testing.assert_array_equal(full[f][i], ref[f][0], err_msg=f"{i} {f}")
    st = cg.stats_dict(out.stats_np())
    assert st["traces"] == N and st["events"] == N * w.events_per_trace()
    assert st["flag_count"] == [0] * 8
    assert st["digest_sum"] == int(s["digest"].astype(np.uint64).sum(dtype=np.uint64))
    rd = out.range_digest.cpu().numpy().view(np.uint64)
    assert int(rd.sum(dtype=np.uint64)) == st["digest_sum"]
    ref = orc.replay_range(w, policy, 5 * rs, 6 * rs)
    assert int(rd[5]) == int(ref["digest"].sum(dtype=np.uint64))


def test_lane16_rejects_unsupported_shapes(cg):
    w = W.CONFIGS["c1"]  # n = 16
    tr = cg.generate(w.gen, 0, 64)
    with pytest.raises(cg.ConvgpuError):
        cg.replay(tr, w.cap, "fifo", cg.alloc_out(64, 16), kernel="lane16")
    w2 = W.CONFIGS["c2"]
    tr = cg.generate(w2.gen, 0, 64)
    with pytest.raises(cg.ConvgpuError):  # neither admit_tick nor the admission scratch
        cg.replay(tr, w2.cap, "fifo", cg.alloc_out(64, 64, full=False, scratch=False),
                  kernel="lane16")
    with pytest.raises(cg.ConvgpuError):  # R1-LIT is not on the 32-bit lane kernel
        cg.replay(tr, w2.cap, "fifo+literal", cg.alloc_out(64, 64), kernel="lane")


def _fused_arrival_batch(seed, count, cap, ovh):
    """Input recipe aimed at the compact kernel's fused arrival step (an
    arrival and its first op applied together when d_0 = 0): many arrivals
    at the same tick, d_0 = 0 for 90 % of containers, first ops of every kind
    with sizes at the boundaries (0, 1, the limit, one over it), limits 0 and
    cap included, and a small capacity so arrivals find a partial target, no
    target with free = 0, or a full ledger."""
    rng = np.random.default_rng(seed)
    n, K = 64, 4
    arrival = np.cumsum(rng.choice([0, 0, 0, 1, 2], size=(count, n)), axis=1).astype(np.uint32)
    lim_menu = np.array([0, 1, cap // 8, cap // 4, cap // 2, cap - 1, cap], np.int64)
    limit = np.where(rng.random((count, n)) < 0.7, lim_menu[rng.integers(0, len(lim_menu), (count, n))],
                     rng.integers(0, cap + 1, (count, n))).astype(np.uint32)
    delta = rng.integers(0, 6, (count, K, n)).astype(np.uint32)
    delta[:, 0, :] = np.where(rng.random((count, n)) < 0.9, 0, rng.integers(1, 4, (count, n)))
    arg = np.zeros((count, K, n), np.uint32)
    for i in range(count):
        bad = rng.random() < 0.1  # this trace may free more than it holds
        for c in range(n):
            L = int(limit[i, c])
            used = 0
            for k in range(K - 1):
                r = rng.random()
                if r < 0.6:
                    room = max(L - ovh - used, 0)
                    sz = int(rng.choice([0, 1, room, room + 1, room // 2, int(rng.integers(0, room + 1))]))
                    kind = W.ALLOC
                    used += sz if sz <= room else 0
                elif r < 0.75:
                    sz = int(rng.choice([0, 1, used, used + 1] if bad else [0, used // 2, used]))
                    sz = sz if (bad or sz <= used) else used
                    kind = W.FREE
                    used -= min(sz, used)
                else:
                    sz, kind = 0, W.NOP
                arg[i, k, c] = W.op(kind, sz)
            arg[i, K - 1, c] = W.op(W.FINISH)
    return W.Batch(n, K, arrival, limit, delta, arg)


@pytest.mark.parametrize("policy", POLS)
@pytest.mark.parametrize("cap,ovh", [(64, 0), (200, 3), (1000, 0)])
def test_lane16_fused_arrival_step(cg, orc, policy, cap, ovh):
    """Element-by-element parity on traces built to hit every branch of the
    fused arrival step: grant / reject / pause (as the new partial target, as
    a zero-assignment newcomer behind a target, and with no target and free =
    0, which triggers a selection), FREE at arrival (0 = valid, 1 = the
    INVALID_FREE stop), NOP, zero limits (admitted on arrival with nothing
    assigned) and same-tick arrival runs."""
    b = _fused_arrival_batch(900 + cap + ovh, 600, cap, ovh)
    base = 123_456_789 + cap
    ref = orc.replay_batch(b, cap, policy, tid_base=base, rand_seed=17 + cap, ovh=ovh)
    tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg, trace_id_base=base)
    out = _gpu_replay(cg, tr, cap, policy, seed=17 + cap, ovh=ovh, kernel="lane16")
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])
    # the batch must exercise the cases it is meant for
    flags = ref["flags"]
    assert (flags & 8).any() and (flags == 0).sum() > 100
    assert int(ref["stats"]["n_select"]) > 0 and int(ref["stats"]["n_rejected"]) > 0


@pytest.mark.parametrize("policy", POLS)
def test_lane16_summary_only_with_scratch(cg, orc, policy):
    """Summary / stats / digest-only launches (no per-container outputs) run on
    the compact kernel through the caller's admission scratch (ABI 4): config
    [2] traces, rho = 8 traces (all through the marked 32-bit fallback) and
    edge-case traces, each against the oracle's summaries and statistics."""
    cases = []
    w = W.CONFIGS["c2"]
    cases.append((w.cap, 0, w.rand_seed, 5_000_000_000, cg.generate(w.gen, 5_000_000_000, 3_001),
                  orc.replay_range(w, policy, 5_000_000_000, 5_000_003_001)))
    w8 = W.rho_sweep(8, rand_seed=9)
    cases.append((w8.cap, 0, 9, 0, cg.generate(w8.gen, 0, 700), orc.replay_range(w8, policy, 0, 700)))
    b = W.random_batch(77, 600, 64, 4, 300, ovh=5, mode="mixed", limit_choices=range(0, 301))
    cases.append((300, 5, 4, 17, cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg,
                                                       trace_id_base=17),
                  orc.replay_batch(b, 300, policy, tid_base=17, rand_seed=4, ovh=5)))
    for cap, ovh, seed, _, tr, ref in cases:
        for kernel in ("lane16", "auto"):
            out = _gpu_replay(cg, tr, cap, policy, seed=seed, ovh=ovh, full=False, kernel=kernel)
            assert out.admit_scratch is not None and out.admit_tick is None
            _compare(cg, out, ref, full=False)
            _compare_stats(cg, out, ref["stats"])


@pytest.mark.parametrize("policy", POLS)
def test_lane16_scratch_reuse_clears_stale_marks(cg, orc, policy):
    """A scratch buffer reused across calls: the first call leaves fallback
    marks (deltas above 16 bits: neither compact layout holds them) in the
    scratch; the second call's traces must not be replayed a second time by a
    fallback pass."""
    import torch
    N = 512
    b0 = W.random_batch(5, N, 64, 4, 200, mode="valid", limit_choices=range(0, 201))
    delta = b0.delta.copy()
    delta[::2, 1, 0] = 0x10000
    tr0 = cg.traces_from_numpy(b0.arrival, b0.limit, delta, b0.arg)
    scratch = torch.empty(N, 64, dtype=torch.int32, device="cuda")
    out = cg.alloc_out(N, 64, full=False, scratch=False)
    out.admit_scratch = scratch
    cg.replay(tr0, 200, policy, out, rand_seed=1, kernel="lane16")
    torch.cuda.synchronize()
    assert (scratch[:, 0].cpu().numpy().view(np.uint32) == 0xFFFFFFFD).any()
    b = W.random_batch(3, N, 64, 4, 200, mode="biglimit", limit_choices=range(0, 201))
    tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg)
    ref = orc.replay_batch(b, 200, policy)
    out2 = cg.alloc_out(N, 64, full=False, scratch=False)
    out2.admit_scratch = scratch
    cg.replay(tr, 200, policy, out2, kernel="lane16")
    torch.cuda.synchronize()
    _compare(cg, out2, ref, full=False)
    _compare_stats(cg, out2, ref["stats"])


CLASS_EDGE = [  # (cap, ovh, mode, count, distinct limits)
    (256, 0, "valid", 700, 8),
    (300, 5, "mixed", 700, 6),
    (200, 1, "delayed", 500, 3),
    (128, 0, "over", 500, 8),
    (256, 0, "badfree", 400, 7),
    (256, 0, "valid", 400, 9),   # one class too many: every trace goes to the fallback
    (256, 2, "valid", 400, 1),   # all limits equal: Best-Fit = FIFO
]


@pytest.mark.parametrize("case", CLASS_EDGE, ids=lambda c: f"{c[2]}{c[0]}o{c[1]}k{c[4]}")
@pytest.mark.parametrize("policy", POLS)
def test_lane16_few_distinct_limits(cg, orc, policy, case):
    """Edge-case programs over a handful of distinct limits, so that Best-Fit
    traces stay on the compact kernel (its limit classes hold <= 8 distinct
    limits; 9 sends the trace to the 32-bit fallback), element by element
    against the oracle.  Limits include 0 and the capacity."""
    cap, ovh, mode, count, k = case
    rng = np.random.default_rng(31 * cap + k)
    menu = ([0] + sorted(int(x) for x in rng.choice(np.arange(1, cap), size=k - 2, replace=False))
            + [cap]) if k >= 2 else [cap // 2]
    b = W.random_batch(5150 + cap + k, count, 64, 4, cap, ovh=ovh, mode=mode,
                       limit_choices=menu)
    base = 3_000_000_000 + cap * k
    ref = orc.replay_batch(b, cap, policy, tid_base=base, rand_seed=9 + k, ovh=ovh)
    tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg, trace_id_base=base)
    out = _gpu_replay(cg, tr, cap, policy, seed=9 + k, ovh=ovh, kernel="lane16")
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])
    if mode in ("valid", "delayed", "over"):
        assert int(ref["stats"]["n_select"]) > 0


# ---------------------------------------------------------------- NEXT-1 on the compact kernel
@pytest.mark.parametrize("policy", POLS)
@pytest.mark.parametrize("rho", [2, 5, 8])
def test_lane16_literal_rho_sweep(cg, orc, policy, rho):
    """R1-LIT (literal re-select-on-every-release, partial holds kept) on the
    compact kernel against the oracle on config [4] traces, element by
    element, including the traces it deadlocks (rho 5: a few; rho = 8: limits
    above 16 bits, so every trace takes the warp-kernel fallback pass)."""
    w = W.rho_sweep(rho, rand_seed=rho + 3)
    pid = POLS.index(policy) | 0x100
    ref = orc.replay_range(w, pid, 20_000, 21_500, full=True)
    tr = cg.generate(w.gen, 20_000, 1_500)
    out = _gpu_replay(cg, tr, w.cap, policy + "+literal", seed=w.rand_seed, kernel="lane16")
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])
    out2 = _gpu_replay(cg, tr, w.cap, policy + "+literal", seed=w.rand_seed, full=False,
                       kernel="lane16")
    _compare(cg, out2, ref, full=False)


LIT_EDGE = [  # (cap, ovh, mode, count)
    (256, 0, "valid", 700),
    (300, 5, "mixed", 900),
    (128, 0, "over", 500),
    (200, 1, "delayed", 500),
    (512, 66, "valid", 500),
]


@pytest.mark.parametrize("case", LIT_EDGE, ids=lambda c: f"{c[2]}{c[0]}o{c[1]}")
@pytest.mark.parametrize("policy", POLS)
def test_lane16_literal_edge_batches(cg, orc, policy, case):
    """R1-LIT on edge-case programs (delayed first ops, rejections, invalid
    frees, bad programs, same-tick arrivals) with dense contention, so many
    containers hold partial assignments and some traces deadlock."""
    cap, ovh, mode, count = case
    b = W.random_batch(8800 + cap, count, 64, 4, cap, ovh=ovh, mode=mode, max_arrival_step=1,
                       limit_choices=range(1, cap + 1))
    pid = POLS.index(policy) | 0x100
    base = 55_000_000 + cap
    ref = orc.replay_batch(b, cap, pid, tid_base=base, rand_seed=6, ovh=ovh)
    tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg, trace_id_base=base)
    out = _gpu_replay(cg, tr, cap, policy + "+literal", seed=6, ovh=ovh, kernel="lane16")
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])
    if mode == "valid":
        assert ref["stats"]["flag_count"][0] > 0  # the literal reading does deadlock here


@pytest.mark.parametrize("policy", POLS)
def test_lane16_literal_mixed_fallback(cg, orc, policy):
    """A batch mixing compact-eligible traces with traces whose values exceed
    the 16-bit fields: the latter are replayed by the warp-per-trace kernel's
    marked-only pass under R1-LIT; every trace against the oracle."""
    xb, cap, ovh = _extreme_batch(97, 300, 64, 4)
    sb = W.random_batch(98, 300, 64, 4, 16, ovh=1, mode="mixed", limit_choices=range(1, 17))
    mix = W.Batch(64, 4, *(np.concatenate([getattr(sb, f), getattr(xb, f)])[np.argsort(
        np.arange(600) % 5, kind="stable")] for f in ("arrival", "limit", "delta", "arg")))
    pid = POLS.index(policy) | 0x100
    ref = orc.replay_batch(mix, cap, pid, tid_base=31, rand_seed=7, ovh=ovh)
    tr = cg.traces_from_numpy(mix.arrival, mix.limit, mix.delta, mix.arg, trace_id_base=31)
    out = _gpu_replay(cg, tr, cap, policy + "+literal", seed=7, ovh=ovh, kernel="lane16")
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])


def _boundary_batch(seed):
    """Traces at the edges of the compact kernel's 16-bit fields and horizon:
    limits 0xFFFE (fits) / 0xFFFF (does not), deltas 0xFFFF / 0x10000, op
    sizes 0xFFFF / 0x10000 (above every 16-bit limit: rejected either way),
    horizons 2^25 - 1 / 2^25 (compact) and 2^26 - 1 / 2^26 (TICK_RANGE), on a
    capacity of 2^26 - 1 MiB.  Each trace's other values are small."""
    rng = np.random.default_rng(seed)
    n, K = 64, 4
    base = W.random_batch(seed, 48, n, K, 200, ovh=3, mode="valid", limit_choices=range(4, 201))
    arrival, limit = base.arrival.copy(), base.limit.copy()
    delta, arg = base.delta.copy(), base.arg.copy()
    cases = []
    for i in range(48):
        c = int(rng.integers(0, n))
        kind = i % 8
        if kind == 0:
            limit[i, c] = 0xFFFE
        elif kind == 1:
            limit[i, c] = 0xFFFF
        elif kind == 2:
            delta[i, 1, c] = 0xFFFF
        elif kind == 3:
            delta[i, 1, c] = 0x10000
        elif kind == 4:
            arg[i, 0, c] = W.op(W.ALLOC, 0xFFFF)
        elif kind == 5:
            arg[i, 0, c] = W.op(W.ALLOC, 0x10000)
        else:  # horizon = max arrival + sum of deltas
            h = int(arrival[i].max()) + int(delta[i].astype(np.uint64).sum())
            target = (1 << 25) - 1 if kind == 6 else (1 << 25)
            if i % 16 >= 8:
                target = (1 << 26) - 1 if kind == 6 else (1 << 26)
            # the last container arrives late enough that the horizon hits the
            # target exactly (arrivals stay sorted, every delta stays small)
            arrival[i, n - 1] += np.uint32(target - h)
        cases.append(kind)
    return W.Batch(n, K, arrival, limit, delta, arg), cases


@pytest.mark.parametrize("policy", POLS)
def test_lane16_field_boundaries(cg, orc, policy):
    """Every boundary of the compact layout against the oracle, element by
    element: values that fit are replayed by the compact kernel, the others by
    the marked fallback pass, and the TICK_RANGE traces are flagged, with the
    same outputs either way."""
    b, _ = _boundary_batch(404)
    cap = (1 << 26) - 1
    ref = orc.replay_batch(b, cap, policy, tid_base=77, rand_seed=5, ovh=3)
    tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg, trace_id_base=77)
    for kernel, full in (("lane16", True), ("lane16", False), ("lane", True), ("warp", True)):
        out = _gpu_replay(cg, tr, cap, policy, seed=5, ovh=3, kernel=kernel, full=full)
        _compare(cg, out, ref, full=full)
        _compare_stats(cg, out, ref["stats"])
    flags = ref["flags"]
    assert (flags & (1 << 5)).any() and (flags == 0).sum() > 20  # TICK_RANGE present, most valid


def _wide_batch(seed):
    """Traces for the compact kernel's 17-bit pass (limits above 0xFFFE): per
    trace i, by i % 8, a few containers get
      0: nothing (16-bit layout)
      1: limit 0x1FFFF, ALLOC 0xFFFE, ALLOC 0xFFFE, FREE 0xFFFE (used reaches
         0x1FFFE with the context charge: the 17-bit used field)
      2: limit 0x10000, ALLOC 0x8000, ALLOC 0x7FFE, FREE 0x8000 (17-bit)
      3: as 1 with a second ALLOC of 0xFFFF (a size above 16 bits: 32-bit pass)
      4: limit 0x20000 (above 17 bits: 32-bit pass)
      5: as 1 with FREE 0xFFFF (32-bit pass)
      6: limit 0x18000, ALLOC 0xFFFE, ALLOC 0xFFFE (the second rejected), FREE
         0x100 (17-bit)
      7: limit 0x1FFFF, first op a FREE of 0xFFFE (INVALID_FREE, 17-bit)
    on a capacity of 0x30000 MiB (the large containers contend), ovh 2."""
    n, K, cap, ovh = 64, 4, 0x30000, 2
    rng = np.random.default_rng(seed)
    # at most 5 distinct limits per trace: Best-Fit's class rule keeps the
    # trace in the compact kernel
    b = W.random_batch(seed, 64, n, K, cap, ovh=ovh, mode="valid", limit_choices=[300, 4000, 9000, 17000])
    limit, arg = b.limit.copy(), b.arg.copy()
    A, F, X = W.ALLOC, W.FREE, W.FINISH
    progs = {1: (0x1FFFF, [(A, 0xFFFE), (A, 0xFFFE), (F, 0xFFFE)]),
             2: (0x10000, [(A, 0x8000), (A, 0x7FFE), (F, 0x8000)]),
             3: (0x1FFFF, [(A, 0xFFFE), (A, 0xFFFF), (F, 0xFFFE)]),
             4: (0x20000, [(A, 0xFFFE), (A, 0xFFFE), (F, 0xFFFE)]),
             5: (0x1FFFF, [(A, 0xFFFE), (A, 0xFFFE), (F, 0xFFFF)]),
             6: (0x18000, [(A, 0xFFFE), (A, 0xFFFE), (F, 0x100)]),
             7: (0x1FFFF, [(F, 0xFFFE), (A, 0x10), (A, 0x10)])}
    for i in range(64):
        kind = i % 8
        if kind == 0:
            continue
        L, prog = progs[kind]
        for c in rng.choice(n, size=6, replace=False):
            limit[i, c] = L
            for k, (kk, sz) in enumerate(prog):
                arg[i, k, c] = W.op(kk, sz)
            arg[i, 3, c] = W.op(X)
    return W.Batch(n, K, b.arrival, limit, b.delta, arg), cap, ovh


@pytest.mark.parametrize("policy", POLS)
def test_lane16_wide_pass(cg, orc, policy):
    """The 17-bit second pass of the compact kernel against the oracle,
    element by element (every kernel variant), and its routing: after a
    summary-only compact replay, exactly the traces the 17-bit layout cannot
    hold carry the second mark (0xFFFFFFFD) in their scratch slot."""
    import torch
    b, cap, ovh = _wide_batch(4242)
    ref = orc.replay_batch(b, cap, policy, tid_base=9, rand_seed=3, ovh=ovh)
    tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg, trace_id_base=9)
    for kernel, full in (("lane16", True), ("lane16", False), ("lane16w", True), ("lane16w", False),
                         ("auto", True), ("lane", True), ("warp", True)):
        out = _gpu_replay(cg, tr, cap, policy, seed=3, ovh=ovh, kernel=kernel, full=full)
        _compare(cg, out, ref, full=full)
        _compare_stats(cg, out, ref["stats"])
    scratch = torch.zeros(64, 64, dtype=torch.int32, device="cuda")
    out = cg.alloc_out(64, 64, full=False, scratch=False)
    out.admit_scratch = scratch
    cg.replay(tr, cap, policy, out, rand_seed=3, ovh=ovh, kernel="lane16")
    torch.cuda.synchronize()
    m2 = scratch[:, 0].cpu().numpy().view(np.uint32) == 0xFFFFFFFD
    kinds = np.arange(64) % 8
    np.testing.assert_array_equal(m2, np.isin(kinds, [3, 4, 5]))
    assert (ref["flags"][kinds == 7] & (1 << 3)).all()  # INVALID_FREE on the 17-bit pass
    assert ref["stats"]["n_rejected"] > 0


@pytest.mark.parametrize("kernel", ["lane16", "lane16w"])
def test_lane16_host_path_wide(cg, orc, kernel):
    """The 32-bit host path (convgpu_replay_host) on config [4] at rho = 8
    (limits above 16 bits) with the compact kernel's 16-bit-first and
    17-bit-first chains: every trace's summary and the statistics of all four
    policies against the oracle."""
    w = W.rho_sweep(8, rand_seed=11)
    base, N = 70_000, 2 * 4096 + 777
    A, L, D, R = orc.generate_batch(w.gen, base, N)
    summ = np.zeros((4, N), cg.SUMMARY_DTYPE)
    st = cg.replay_host(A, L, D, R, w.cap, POLS, trace_id_base=base, summary=summ,
                        rand_seed=11, chunk=4096, kernel=kernel)
    for q, pol in enumerate(POLS):
        ref = orc.replay_range(w, pol, base, base + N)
        for f in ("makespan", "peak_reserved", "peak_used", "flags", "sum_wait", "n_rejected",
                  "n_select", "digest"):
            np.testing.assert_array_equal(summ[q][f], ref[f].astype(summ[q][f].dtype),
                                          err_msg=f"{pol} {f}")
        for k, v in ref["stats"].items():
            assert cg.stats_dict(st[q])[k] == v, (pol, k)


def _off16(t, torch):
    """A contiguous copy of `t` whose data starts 16 bytes past a 32-byte
    boundary (16-B aligned, not 32-B aligned)."""
    es = t.element_size()
    big = torch.empty(t.numel() + 64 // es, dtype=t.dtype, device=t.device)
    base = big.data_ptr()
    skip = ((32 - base % 32) % 32 + 16) // es
    v = big[skip:skip + t.numel()].view(t.shape)
    v.copy_(t)
    assert v.data_ptr() % 32 == 16
    return v


@pytest.mark.parametrize("policy", POLS)
@pytest.mark.parametrize("which", ["traces", "outputs"])
def test_lane16_16byte_aligned_path(cg, orc, policy, which):
    """Arrays 16-B but not 32-B aligned take the compact kernel's 16-byte
    init / epilogue path (the 32-byte one needs every trace array and output
    32-B aligned): config [2] traces, full outputs and summary-only through
    the admission scratch, against the oracle."""
    import torch
    w = W.CONFIGS["c2"]
    base, N = 123_456, 5_000
    tr0 = cg.generate(w.gen, base, N)
    tr = tr0
    if which == "traces":
        tr = cg.Traces(_off16(tr0.arrival, torch), _off16(tr0.limit, torch),
                       _off16(tr0.op_delta, torch), _off16(tr0.op_arg, torch), base)
    ref = orc.replay_range(w, policy, base, base + N, full=True)
    out = cg.alloc_out(N, 64)
    if which == "outputs":
        out.admit_tick = _off16(out.admit_tick, torch)
        out.wait = _off16(out.wait, torch)
        out.finish = _off16(out.finish, torch)
    cg.replay(tr, w.cap, policy, out, rand_seed=w.rand_seed, kernel="lane16")
    torch.cuda.synchronize()
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])
    outs = cg.alloc_out(N, 64, full=False)
    if which == "outputs":
        outs.admit_scratch = _off16(outs.admit_scratch, torch)
    cg.replay(tr, w.cap, policy, outs, rand_seed=w.rand_seed, kernel="lane16")
    torch.cuda.synchronize()
    _compare(cg, outs, ref, full=False)
    _compare_stats(cg, outs, ref["stats"])
