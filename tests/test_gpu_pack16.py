"""The compact 16-bit host format (include/convgpu.h convgpu_traces16_t):
convgpu_pack16 against a numpy packing of the same arrays (the definition:
each field's low 16 bits, kinds 2 bits per op), its out-of-range count, and
convgpu_replay_host16 end to end against the oracle and against the 32-bit
host path, bit for bit.  Needs a B200."""
import numpy as np
import pytest

import workloads as W
from test_gpu_parity import SUMMARY_FIELDS

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cg():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_cluster_kangjkkk17_b200 as m
    from paper_conf_cluster_kangjkkk17_b200 import build
    build.build()
    return m


def _np_pack(A, L, D, R):
    """Reference packing in numpy (definition of the format)."""
    K = D.shape[1]
    kinds = np.zeros(A.shape, np.uint32)
    for k in range(K):
        kinds |= (R[:, k, :] >> 30) << (2 * k)
    return ((A & 0xFFFF).astype(np.uint16), (L & 0xFFFF).astype(np.uint16),
            (R & 0xFFFF).astype(np.uint16), (D & 0xFFFF).astype(np.uint16), kinds.astype(np.uint8))


def _host(cg, t):
    return [x.cpu().numpy().view(np.uint32) for x in (t.arrival, t.limit, t.op_delta, t.op_arg)]


@pytest.mark.parametrize("case", ["c2", "mimic", "edge"])
def test_pack16_matches_numpy_definition(cg, case):
    import torch
    if case == "edge":
        b = W.random_batch(71, 900, 13, 4, 300, ovh=3, mode="mixed",
                           limit_choices=range(0, 301))
        tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg)
    else:
        w = W.CONFIGS[case]
        tr = cg.generate(w.gen, 12_345, 3_001)
    t16, oor = cg.pack16(tr)
    torch.cuda.synchronize()
    A, L, D, R = _host(cg, tr)
    want = _np_pack(A, L, D, R)
    have = [t16.arrival, t16.limit, t16.op_size, t16.op_delta, t16.op_kinds]
    for h, x in zip(have, want):
        np.testing.assert_array_equal(h.cpu().numpy().view(x.dtype), x)
    n_big = int((A > 0xFFFF).sum() + (L > 0xFFFF).sum() + ((R & 0x3FFFFFFF) > 0xFFFF).sum() +
                (D > 0xFFFF).sum())
    assert int(oor.item()) == n_big


def test_pack16_counts_out_of_range(cg):
    import torch
    w = W.rho_sweep(8)  # limits up to 70,217 MiB: some exceed 16 bits
    tr = cg.generate(w.gen, 0, 2_000)
    _, oor = cg.pack16(tr)
    torch.cuda.synchronize()
    A, L, D, R = _host(cg, tr)
    want = int((L > 0xFFFF).sum() + ((R & 0x3FFFFFFF) > 0xFFFF).sum())
    assert want > 0 and int(oor.item()) == want


@pytest.mark.parametrize("chunk", [1024, 4096])
def test_replay_host16_end_to_end(cg, orc, chunk):
    """All four policies from 16-bit pinned host traces: every summary field
    against the oracle, and the statistics equal the 32-bit host path's."""
    w = W.CONFIGS["c2"]
    N = 5_000
    base = 777_000
    tr = cg.generate(w.gen, base, N)
    t16, oor = cg.pack16(tr)
    assert int(oor.item()) == 0
    h16 = t16.pin()
    summ = np.zeros((4, N), cg.SUMMARY_DTYPE)
    st = cg.replay_host16(h16, w.cap, W.POLICIES, trace_id_base=base, rand_seed=3, chunk=chunk,
                          summary=summ)
    A, L, D, R = _host(cg, tr)
    summ32 = np.zeros((4, N), cg.SUMMARY_DTYPE)
    st32 = cg.replay_host(A, L, D, R, w.cap, W.POLICIES, trace_id_base=base, rand_seed=3,
                          chunk=chunk, summary=summ32)
    for q, pol in enumerate(W.POLICIES):
        ref = orc.replay_range(w, pol, base, base + N, rand_seed=3)
        for f in SUMMARY_FIELDS:
            np.testing.assert_array_equal(summ[q][f], ref[f].astype(summ[q][f].dtype), err_msg=f)
        for k, v in ref["stats"].items():
            assert cg.stats_dict(st[q])[k] == v, (pol, k)
        assert cg.stats_dict(st[q]) == cg.stats_dict(st32[q])
    assert (summ == summ32).all()


@pytest.mark.parametrize("policy", ["fifo", "best_fit", "recent_fit", "random_fit"])
def test_replay_host16_edge_batches(cg, orc, policy):
    """Edge-case traces (n = 13, ragged; every op kind, rejections, invalid
    frees, bad programs) through the 16-bit host path, against the oracle."""
    b = W.random_batch(72, 1_500, 13, 4, 300, ovh=3, mode="mixed", limit_choices=range(0, 301))
    tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg)
    t16, oor = cg.pack16(tr)
    assert int(oor.item()) == 0
    summ = np.zeros((1, b.count), cg.SUMMARY_DTYPE)
    st = cg.replay_host16(t16.pin(), 300, (policy,), trace_id_base=40, rand_seed=8, ovh=3,
                          chunk=333, summary=summ)
    ref = orc.replay_batch(b, 300, policy, tid_base=40, rand_seed=8, ovh=3)
    for f in SUMMARY_FIELDS:
        np.testing.assert_array_equal(summ[0][f], ref[f].astype(summ[0][f].dtype), err_msg=f)
    for k, v in ref["stats"].items():
        assert cg.stats_dict(st[0])[k] == v, (policy, k)


@pytest.mark.parametrize("policy", ["fifo", "best_fit", "recent_fit", "random_fit"])
def test_replay_host16_other_shapes(cg, orc, policy):
    """The 16-bit host path with K = 2 (paper-mimic programs, n = 38, 66-MiB
    context; arrivals 500 ticks apart so that they fit 16 bits — the paper's
    5,000-tick spacing does not, and pack16 counts it) and K = 1
    (FINISH-only programs, n = 5): summaries and stats vs the oracle."""
    import dataclasses
    w = W.CONFIGS["mimic"]
    tr = cg.generate(w.gen, 3_000, 100)
    _, oor = cg.pack16(tr)
    assert int(oor.item()) == 100 * 24  # arrivals 5,000 x c > 0xFFFF for c = 14 .. 37
    w = dataclasses.replace(w, gen=dataclasses.replace(w.gen, iat=500))
    tr = cg.generate(w.gen, 3_000, 2_500)
    t16, oor = cg.pack16(tr)
    assert int(oor.item()) == 0
    summ = np.zeros((1, 2_500), cg.SUMMARY_DTYPE)
    st = cg.replay_host16(t16.pin(), w.cap, (policy,), trace_id_base=3_000, rand_seed=w.rand_seed,
                          ovh=w.ovh, chunk=700, summary=summ)
    ref = orc.replay_range(w, policy, 3_000, 5_500)
    for f in SUMMARY_FIELDS:
        np.testing.assert_array_equal(summ[0][f], ref[f].astype(summ[0][f].dtype), err_msg=f)
    for k, v in ref["stats"].items():
        assert cg.stats_dict(st[0])[k] == v, (policy, k)
    b = W.random_batch(74, 600, 5, 1, 40, mode="valid", limit_choices=range(0, 41))
    tr = cg.traces_from_numpy(b.arrival, b.limit, b.delta, b.arg)
    t16, oor = cg.pack16(tr)
    summ = np.zeros((1, 600), cg.SUMMARY_DTYPE)
    st = cg.replay_host16(t16.pin(), 40, (policy,), chunk=256, summary=summ)
    ref = orc.replay_batch(b, 40, policy)
    for f in SUMMARY_FIELDS:
        np.testing.assert_array_equal(summ[0][f], ref[f].astype(summ[0][f].dtype), err_msg=f)
