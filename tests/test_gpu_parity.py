"""GPU parity: the CUDA path (through the C ABI) against the C oracle,
element by element, bit-exact on every integer field (BASELINE.json
north_star).  Needs a B200: run via gpurun."""
import numpy as np
import pytest

import workloads as W

pytestmark = pytest.mark.gpu
POLS = ["fifo", "best_fit", "recent_fit", "random_fit"]
SUMMARY_FIELDS = ["makespan", "peak_reserved", "peak_used", "flags", "sum_wait", "n_rejected",
                  "n_select", "digest"]


@pytest.fixture(scope="module")
def cg():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_cluster_kangjkkk17_b200 as m
    from paper_conf_cluster_kangjkkk17_b200 import build
    build.build()
    return m


KERNELS = ["warp", "lane"]


def _gpu_replay(cg, tr, cap, policy, seed=0, ovh=0, full=True, range_size=0, range_count=0,
                kernel="auto", scratch=None):
    import torch
    out = cg.alloc_out(tr.count, tr.n, full=full, range_count=range_count,
                       range_size=range_size, scratch=scratch)
    cg.replay(tr, cap, policy, out, rand_seed=seed, ovh=ovh, kernel=kernel)
    torch.cuda.synchronize()
    return out


def _compare(cg, out, ref, idx=None, full=True):
    s = out.summary_np()
    if idx is not None:
        s = s[idx]
    for f in SUMMARY_FIELDS:
        np.testing.assert_array_equal(s[f], ref[f].astype(s[f].dtype), err_msg=f)
    if full:
        g = out.full_np()
        for f in ("admit_tick", "admit_rank", "wait", "finish"):
            a = g[f] if idx is None else g[f][idx]
            np.testing.assert_array_equal(a, ref[f], err_msg=f)


def _compare_stats(cg, out, ref_stats):
    st = cg.stats_dict(out.stats_np())
    for k, v in ref_stats.items():
        assert st[k] == v, (k, st[k], v)


# ---------------------------------------------------------------- generator
@pytest.mark.parametrize("cfg", ["c1", "c2", "mimic"])
def test_generator_bit_exact(cg, orc, cfg):
    w = W.CONFIGS[cfg]
    base, count = 123_456_789_000, 777
    t = cg.generate(w.gen, base, count)
    A, L, D, R = orc.generate_batch(w.gen, base, count)
    np.testing.assert_array_equal(t.arrival.cpu().numpy().view(np.uint32), A)
    np.testing.assert_array_equal(t.limit.cpu().numpy().view(np.uint32), L)
    np.testing.assert_array_equal(t.op_delta.cpu().numpy().view(np.uint32), D)
    np.testing.assert_array_equal(t.op_arg.cpu().numpy().view(np.uint32), R)


def test_generator_jitter_and_64bit_ids(cg, orc):
    g = W.GenParams(n=37, K=4, class_mib=(100, 7000, 33), num=5, den=3, iat=17, dur_jit=999,
                    dur_class_offset=1, ovh=66, gen_seed=0xDEADBEEFCAFEF00D)
    base = (1 << 40) - 100
    t = cg.generate(g, base, 300)
    A, L, D, R = orc.generate_batch(g, base, 300)
    np.testing.assert_array_equal(t.op_delta.cpu().numpy().view(np.uint32), D)
    np.testing.assert_array_equal(t.op_arg.cpu().numpy().view(np.uint32), R)
    np.testing.assert_array_equal(t.limit.cpu().numpy().view(np.uint32), L)


# ---------------------------------------------------------------- replay
@pytest.mark.parametrize("policy", POLS)
@pytest.mark.parametrize("kernel", KERNELS)
def test_fig3_on_gpu(cg, orc, kernel, policy):
    from conftest import golden
    f = W.fig3_fixture()
    tr = cg.traces_from_numpy(f["arrival"][None], f["limit"][None], f["delta"][None],
                              f["arg"][None])
    out = _gpu_replay(cg, tr, f["cap"], policy, kernel=kernel)
    g = golden("fig3.json")["expected_all_policies"]
    s = out.summary_np()[0]
    full = out.full_np()
    assert list(full["admit_tick"][0]) == g["admit_tick"]
    assert list(full["admit_rank"][0]) == g["admit_rank"]
    assert list(full["wait"][0]) == g["wait"]
    assert list(full["finish"][0]) == g["finish"]
    for k in ("makespan", "peak_reserved", "peak_used", "sum_wait", "n_select", "n_rejected", "flags"):
        assert int(s[k]) == g[k], k
    assert cg.stats_dict(out.stats_np())["events"] == g["events"]


EDGE = [  # (n, K, cap, ovh, mode, count)
    (1, 1, 8, 0, "mixed", 300),
    (3, 2, 8, 0, "valid", 500),
    (4, 3, 8, 0, "delayed", 700),
    (5, 4, 8, 1, "over", 700),
    (7, 5, 16, 2, "mixed", 1000),
    (16, 4, 64, 0, "valid", 1000),
    (31, 6, 100, 3, "mixed", 600),
    (32, 8, 128, 0, "badfree", 600),
    (33, 4, 200, 0, "valid", 600),
    (63, 7, 300, 5, "mixed", 400),
    (64, 8, 256, 0, "over", 400),
    (64, 4, 512, 66, "valid", 400),
]


@pytest.mark.parametrize("case", EDGE, ids=lambda c: f"n{c[0]}K{c[1]}{c[4]}")
@pytest.mark.parametrize("policy", POLS)
@pytest.mark.parametrize("kernel", KERNELS)
def test_edge_batches(cg, orc, kernel, case, policy):
    n, K, cap, ovh, mode, count = case
    b = W.random_batch(1000 + n * 10 + K, count, n, K, cap, ovh=ovh, mode=mode,
                       limit_choices=range(0, cap + 1))
    base = 5_000_000_000 + n
    ref = orc.replay_batch(b, cap, policy, tid_base=base, rand_seed=99 + n, ovh=ovh)
    tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg, trace_id_base=base)
    out = _gpu_replay(cg, tr, cap, policy, seed=99 + n, ovh=ovh, kernel=kernel)
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])


@pytest.mark.parametrize("policy", POLS)
@pytest.mark.parametrize("kernel", KERNELS)
def test_config1_full(cg, orc, kernel, policy):
    """BASELINE config [1]: 10^4 traces x 16 containers, every output field."""
    w = W.CONFIGS["c1"]
    N = w.n_traces
    ref = orc.replay_range(w, policy, 0, N, full=True)
    tr = cg.generate(w.gen, 0, N)
    out = _gpu_replay(cg, tr, w.cap, policy, seed=w.rand_seed, kernel=kernel)
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])
    assert ref["stats"]["flag_count"][0] == 0  # no deadlock (P:7)


@pytest.mark.parametrize("policy", POLS)
@pytest.mark.parametrize("kernel", KERNELS)
def test_config2_window_with_ragged_tail(cg, orc, kernel, policy):
    """Config [2] generator; a window of trace ids whose count is not a
    multiple of the warps in flight, at an unaligned 64-bit base."""
    w = W.CONFIGS["c2"]
    base, N = 987_654_321_001, 4_741
    ref = orc.replay_range(w, policy, base, base + N, full=True)
    tr = cg.generate(w.gen, base, N)
    out = _gpu_replay(cg, tr, w.cap, policy, seed=w.rand_seed, kernel=kernel)
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])


@pytest.mark.parametrize("policy", POLS)
@pytest.mark.parametrize("kernel", KERNELS)
def test_mimic_with_overhead(cg, orc, kernel, policy):
    w = W.CONFIGS["mimic"]
    N = 3000
    ref = orc.replay_range(w, policy, 0, N, full=True)
    tr = cg.generate(w.gen, 0, N)
    out = _gpu_replay(cg, tr, w.cap, policy, seed=w.rand_seed, ovh=w.ovh, kernel=kernel)
    _compare(cg, out, ref)


@pytest.mark.parametrize("policy", POLS)
@pytest.mark.parametrize("rho", [1, 2, 3, 4, 5, 6, 7, 8])
@pytest.mark.parametrize("kernel", KERNELS)
def test_rho_sweep_window(cg, orc, kernel, policy, rho):
    w = W.rho_sweep(rho, rand_seed=rho * 7 + 1)
    ref = orc.replay_range(w, policy, 10_000, 11_000, full=True)
    tr = cg.generate(w.gen, 10_000, 1_000)
    out = _gpu_replay(cg, tr, w.cap, policy, seed=w.rand_seed, kernel=kernel)
    _compare(cg, out, ref)


@pytest.mark.parametrize("policy", POLS)
def test_config2_full_size_sampled(cg, orc, policy):
    """BASELINE config [2] at full size (10^6 traces) in the bench launch
    configuration (summary-only outputs, stats + range digests): sampled
    traces recomputed one by one by the oracle; size-independent properties
    on all of them."""
    import torch
    w = W.CONFIGS["c2"]
    N = w.n_traces
    tr = cg.generate(w.gen, 0, N)
    rs = 1 << 16
    out = _gpu_replay(cg, tr, w.cap, policy, seed=w.rand_seed, full=False, range_size=rs,
                      range_count=(N + rs - 1) // rs)
    s = out.summary_np()
    rng = np.random.default_rng(5)
    idx = np.unique(np.concatenate([rng.integers(0, N, 300), [0, 1, N - 2, N - 1]]))
    for i in idx:
        ref = orc.replay_range(w, policy, int(i), int(i) + 1)
        for f in SUMMARY_FIELDS:
            assert int(s[f][i]) == int(ref[f][0]), (i, f)
    st = cg.stats_dict(out.stats_np())
    assert st["traces"] == N and st["events"] == N * w.events_per_trace()
    assert st["flag_count"] == [0] * 8
    assert st["max_peak_reserved"] <= w.cap
    assert (s["peak_used"] <= s["peak_reserved"]).all()
    assert st["digest_sum"] == int(s["digest"].astype(np.uint64).sum(dtype=np.uint64))
    # one full range digest against the oracle
    ref = orc.replay_range(w, policy, 3 * rs, 4 * rs)
    rd = out.range_digest.cpu().numpy().view(np.uint64)
    assert int(rd[3]) == int(ref["digest"].sum(dtype=np.uint64))
    assert int(rd.sum(dtype=np.uint64)) == st["digest_sum"]


def test_bulk_and_plain_staging_agree(cg, orc):
    """n % 4 == 0 with 16-B aligned arrays uses the bulk-copy (TMA) staging;
    an offset view forces the plain-load path: results must be identical."""
    import torch
    w = W.CONFIGS["c2"]
    tr = cg.generate(w.gen, 0, 2000)
    out1 = _gpu_replay(cg, tr, w.cap, "best_fit")
    big = cg.empty_traces(2001, 64, 4)
    for a, b in ((big.arrival, tr.arrival), (big.limit, tr.limit), (big.op_delta, tr.op_delta),
                 (big.op_arg, tr.op_arg)):
        a.view(-1)[1:1 + b.numel()].copy_(b.view(-1))
    mis = cg.Traces(big.arrival.view(-1)[1:1 + tr.arrival.numel()].view(2000, 64),
                    big.limit.view(-1)[1:1 + tr.limit.numel()].view(2000, 64),
                    big.op_delta.view(-1)[1:1 + tr.op_delta.numel()].view(2000, 4, 64),
                    big.op_arg.view(-1)[1:1 + tr.op_arg.numel()].view(2000, 4, 64))
    out2 = _gpu_replay(cg, mis, w.cap, "best_fit")
    assert (out1.summary.cpu() == out2.summary.cpu()).all()


def test_replay_host_end_to_end(cg, orc):
    w = W.CONFIGS["c2"]
    N = 5000
    A, L, D, R = orc.generate_batch(w.gen, 0, N)
    pols = ("best_fit", "recent_fit", "random_fit")
    summ = np.zeros((3, N), cg.SUMMARY_DTYPE)
    st = cg.replay_host(A, L, D, R, w.cap, pols, chunk=1024, summary=summ, rand_seed=5)
    for q, pol in enumerate(pols):
        ref = orc.replay_range(w, pol, 0, N, rand_seed=5)
        for f in SUMMARY_FIELDS:
            np.testing.assert_array_equal(summ[q][f], ref[f].astype(summ[q][f].dtype), err_msg=f)
        for k, v in ref["stats"].items():
            assert cg.stats_dict(st[q])[k] == v, (pol, k)


def test_errors_and_empty(cg):
    import ctypes as C
    import errno
    import torch
    t = cg.generate(W.CONFIGS["c1"].gen, 0, 4)
    out = cg.alloc_out(0, 16)
    empty = cg.Traces(t.arrival[:0], t.limit[:0], t.op_delta[:0], t.op_arg[:0])
    cg.replay(empty, 8192, "fifo", out)  # n == 0 is a no-op
    host = t.arrival.cpu()
    bad = cg.TracesT(host.data_ptr(), t.limit.data_ptr(), t.op_delta.data_ptr(),
                     t.op_arg.data_ptr(), 16, 4, 0, 0, 0, 0)
    o = cg.OutT()
    assert cg.lib().convgpu_replay(C.byref(bad), 4, 8192, 0, C.byref(o)) == -errno.EINVAL
    with pytest.raises(cg.ConvgpuError):
        cg.replay(t, 0, "fifo", cg.alloc_out(4, 16))


def test_stats_accumulate_across_calls_and_streams(cg, orc):
    import torch
    w = W.CONFIGS["c1"]
    tr = cg.generate(w.gen, 0, 3000)
    out = cg.alloc_out(3000, 16, full=False)
    s = torch.cuda.Stream()
    cg.replay(tr, w.cap, "fifo", out, stream=s)
    cg.replay(tr, w.cap, "fifo", out, stream=s)
    s.synchronize()
    ref = orc.replay_range(w, "fifo", 0, 3000)["stats"]
    st = cg.stats_dict(out.stats_np())
    assert st["traces"] == 2 * ref["traces"] and st["events"] == 2 * ref["events"]
    assert st["max_makespan"] == ref["max_makespan"]


# ---------------------------------------------------------------- NEXT-1
@pytest.mark.parametrize("policy", POLS)
@pytest.mark.parametrize("case", [(4, 3, 8, 0, "valid", 2000), (7, 5, 16, 2, "mixed", 1500),
                                  (64, 4, 512, 66, "valid", 400)], ids=["n4", "n7mixed", "n64"])
def test_literal_reading_parity(cg, orc, policy, case):
    """R1-LIT (literal re-select-on-every-release) on the GPU vs the oracle,
    including the traces it deadlocks (flag bit 0, zeroed outputs)."""
    n, K, cap, ovh, mode, count = case
    b = W.random_batch(77 + n, count, n, K, cap, ovh=ovh, mode=mode, max_arrival_step=1,
                       limit_choices=range(1, cap + 1))
    pid = POLS.index(policy) | 0x100
    ref = orc.replay_batch(b, cap, pid, tid_base=9, rand_seed=4, ovh=ovh)
    tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg, trace_id_base=9)
    out = _gpu_replay(cg, tr, cap, policy + "+literal", seed=4, ovh=ovh)
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])


@pytest.mark.parametrize("policy", POLS)
def test_literal_reading_deadlocks_on_paper_mimic(cg, orc, policy):
    """The paper-mimic workload under R1-LIT vs R1 on the GPU:
    the literal reading deadlocks a share of traces, R1 none (P:7)."""
    w = W.CONFIGS["mimic"]
    N = 2000
    tr = cg.generate(w.gen, 0, N)
    lit = _gpu_replay(cg, tr, w.cap, policy + "+literal", seed=w.rand_seed, ovh=w.ovh)
    ref = orc.replay_range(w, POLS.index(policy) | 0x100, 0, N, full=True)
    _compare(cg, lit, ref)
    sticky = _gpu_replay(cg, tr, w.cap, policy, seed=w.rand_seed, ovh=w.ovh, full=False)
    assert cg.stats_dict(sticky.stats_np())["flag_count"][0] == 0


def _extreme_batch(seed, count, n, K):
    """Values at the ABI limits: capacity 2^26-1, limits up to it, ALLOC sizes
    up to 2^30-1 (over-limit ones are rejected), large deltas with trace
    horizons at exactly 2^26-1 (valid) and >= 2^26 (TICK_RANGE)."""
    rng = np.random.default_rng(seed)
    cap = (1 << 26) - 1
    parts = [W.random_batch(seed + j, count // 3, n, K, 16, ovh=1, mode=m, max_arrival_step=2,
                            limit_choices=range(1, 17))
             for j, m in enumerate(("valid", "over", "delayed"))]
    cat = lambda f: np.concatenate([getattr(b, f) for b in parts])  # noqa: E731
    arrival, limit, delta, arg = cat("arrival"), cat("limit"), cat("delta"), cat("arg")
    N = arrival.shape[0]
    scale = cap // 16
    limit = np.minimum(limit.astype(np.uint64) * scale, cap).astype(np.uint32)
    kinds = arg >> 30
    sizes = (arg & 0x3FFFFFFF).astype(np.uint64) * scale
    big = (rng.random(sizes.shape) < 0.05) & (kinds == 0)  # huge ALLOCs: rejected
    sizes = np.where(big, (1 << 30) - 1, np.minimum(sizes, (1 << 30) - 1)).astype(np.uint32)
    arg = ((kinds << 30) | sizes).astype(np.uint32)
    unit = (1 << 26) // (4 * (n * K + 1))
    delta = (delta.astype(np.uint64) * unit).astype(np.uint32)
    arrival = (arrival.astype(np.uint64) * unit).astype(np.uint32)
    for i in range(N):  # horizon = max arrival + sum of deltas
        h = int(arrival[i].max()) + int(delta[i].astype(np.uint64).sum())
        if i % 5 == 0:
            delta[i, K - 1, 0] += np.uint32((1 << 26) - 1 - h)  # exactly representable
        elif i % 5 == 1:
            delta[i, K - 1, 0] += np.uint32((1 << 26) - h)      # one past: TICK_RANGE
    return W.Batch(n, K, arrival, limit, delta, arg), cap, scale  # overhead = 1 unit


@pytest.mark.parametrize("kernel", KERNELS)
@pytest.mark.parametrize("policy", POLS)
@pytest.mark.parametrize("nk", [(8, 4), (64, 8)], ids=["n8K4", "n64K8"])
def test_extreme_values(cg, orc, kernel, policy, nk):
    n, K = nk
    b, cap, ovh = _extreme_batch(31 + n, 300, n, K)
    ref = orc.replay_batch(b, cap, policy, tid_base=2**63 + 5, rand_seed=2**64 - 1, ovh=ovh)
    st = ref["stats"]
    assert st["flag_count"][5] > 0 and st["n_select"] > 0 and st["n_rejected"] > 0
    tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg, trace_id_base=2**63 + 5)
    out = _gpu_replay(cg, tr, cap, policy, seed=2**64 - 1, ovh=ovh, kernel=kernel)
    _compare(cg, out, ref)
    _compare_stats(cg, out, ref["stats"])


def test_replay_host_production_chunks(cg, orc):
    """The host path as bench.py's e2e leg runs it: default 32,768-trace chunks
    (compact lane kernel, two copy streams), a short tail chunk (warp kernel
    below 40 traces per SM), every policy on each resident chunk.  Every
    trace's summary is compared with the oracle's, field by field."""
    w = W.CONFIGS["c2"]
    base, N = 3_000_000, 2 * 32768 + 3001
    A, L, D, R = orc.generate_batch(w.gen, base, N)
    summ = np.zeros((4, N), cg.SUMMARY_DTYPE)
    st = cg.replay_host(A, L, D, R, w.cap, POLS, trace_id_base=base, summary=summ,
                        rand_seed=w.rand_seed)
    for q, pol in enumerate(POLS):
        ref = orc.replay_range(w, pol, base, base + N)
        for f in SUMMARY_FIELDS:
            np.testing.assert_array_equal(summ[q][f], ref[f].astype(summ[q][f].dtype),
                                          err_msg=f"{pol} {f}")
        for k, v in ref["stats"].items():
            assert cg.stats_dict(st[q])[k] == v, (pol, k)
