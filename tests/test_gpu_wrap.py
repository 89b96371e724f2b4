"""NEXT-3 on the GPU: convgpu_wrap_ops (csrc/wrap.cu) against the oracle's
wrapper semantics (oracle/wrapper.c), bit for bit, and end to end through the
replay.  Also pins the kernel live to the CUDA runtime's cudaMallocPitch on
the box it runs on."""
import numpy as np
import pytest

import workloads as W

pytestmark = pytest.mark.gpu


def _dev(api):
    import torch
    a = np.ascontiguousarray(api).view(np.uint32).reshape(api.shape + (4,))
    return torch.from_numpy(a.view(np.int32)).cuda()


def _wrap_gpu(api, pitch=512):
    import torch

    import paper_conf_cluster_kangjkkk17_b200 as cg
    N, K, n = api.shape
    out = cg.wrap_ops(_dev(api), n, K, pitch_align=pitch)
    torch.cuda.synchronize()
    return out.cpu().numpy().view(np.uint32)


@pytest.mark.parametrize("shape", [(2048, 64, 4), (501, 5, 7), (300, 64, 8), (1, 1, 1), (77, 33, 3)])
@pytest.mark.parametrize("mode", ["valid", "mixed"])
def test_wrap_parity(orc, shape, mode):
    N, n, K = shape
    api = W.random_api_batch(hash((shape, mode)) & 0xFFFF, N, n, K, mode)
    for pitch in (512, 0, 1, 32, 1000):
        got = _wrap_gpu(api, pitch)
        want = orc.wrap_batch(api, pitch)
        bad = np.argwhere(got != want)
        assert bad.size == 0, (pitch, bad[:5], got[tuple(bad[0])], want[tuple(bad[0])])


def test_wrap_pitch_matches_the_live_runtime():
    """The kernel's pitched size equals what cudaMallocPitch returns here."""
    from cuda.bindings import runtime as rt
    err, prop = rt.cudaGetDeviceProperties(0)
    A = int(prop.textureAlignment)
    widths = list(range(1, 1200, 7)) + [4095, 4096, 4097, 65535, 65536, 1 << 20]
    api = np.zeros((len(widths), 1, 1), W.API_RECORD)  # one single-op trace per width
    for j, w in enumerate(widths):
        api[j, 0, 0] = (W.API_PITCH, w, 1 << 20, 0)  # 2^20 rows: bytes = pitch MiB exactly
    got = _wrap_gpu(api, A)[:, 0, 0]
    for j, w in enumerate(widths):
        err, ptr, pitch = rt.cudaMallocPitch(w, 1)
        assert err == rt.cudaError_t.cudaSuccess
        rt.cudaFree(ptr)
        assert got[j] == pitch, (w, pitch, got[j])  # ALLOC << 30 is 0


@pytest.mark.parametrize("kernel", ["warp", "lane"])
def test_wrap_then_replay_end_to_end(orc, kernel):
    import torch

    import paper_conf_cluster_kangjkkk17_b200 as cg
    N, n, K = 600, 16, 6
    api = W.random_api_batch(31, N, n, K, "valid", scale_mib=2048)
    api[: N // 5] = W.random_api_batch(33, N // 5, n, K, "mixed", scale_mib=2048)
    rng = np.random.default_rng(32)
    arrival = np.cumsum(rng.integers(0, 40, (N, n)), axis=1).astype(np.uint32)
    limit = rng.integers(0, 8192, (N, n)).astype(np.uint32)
    delta = rng.integers(0, 50, (N, K, n)).astype(np.uint32)
    words = orc.wrap_batch(api, 512)
    tr = cg.traces_from_numpy(arrival, limit, delta, words)
    cg.wrap_ops(_dev(api), n, K, out=tr.op_arg)  # the device's own words replace the oracle's
    for pol in ("fifo", "best_fit", "recent_fit", "random_fit"):
        out = cg.alloc_out(N, n)
        cg.replay(tr, 8192, pol, out, rand_seed=3, kernel=kernel)
        torch.cuda.synchronize()
        b = W.Batch(n, K, arrival, limit, delta, words)
        ref = orc.replay_batch(b, 8192, pol, rand_seed=3)
        s = out.summary_np()
        for f in ("makespan", "peak_reserved", "flags", "digest"):
            assert np.array_equal(s[f], ref[f]), (pol, f)
        full = out.full_np()
        for f in ("admit_tick", "wait", "finish"):
            assert np.array_equal(full[f], ref[f]), (pol, f)
    assert (ref["flags"] & 8).any() and (ref["flags"] & 64).any()  # the mix reaches both flags
    assert (ref["flags"] == 0).mean() > 0.3


def test_wrap_errors_and_empty():
    import torch

    import paper_conf_cluster_kangjkkk17_b200 as cg
    L = cg.lib()
    api = torch.zeros((4, 2, 3, 4), dtype=torch.int32, device="cuda")
    out = torch.zeros((4, 2, 3), dtype=torch.int32, device="cuda")
    s = torch.cuda.current_stream().cuda_stream
    assert L.convgpu_wrap_ops(api.data_ptr(), 4, 3, 2, 512, out.data_ptr(), s) == 0
    assert L.convgpu_wrap_ops(api.data_ptr() + 4, 3, 3, 2, 512, out.data_ptr(), s) < 0  # unaligned
    assert L.convgpu_wrap_ops(api.data_ptr(), 4, 0, 2, 512, out.data_ptr(), s) < 0
    assert L.convgpu_wrap_ops(api.data_ptr(), 4, 65, 2, 512, out.data_ptr(), s) < 0
    assert L.convgpu_wrap_ops(api.data_ptr(), 4, 3, 9, 512, out.data_ptr(), s) < 0
    assert L.convgpu_wrap_ops(None, 4, 3, 2, 512, out.data_ptr(), s) < 0
    assert L.convgpu_wrap_ops(None, 0, 3, 2, 512, None, s) == 0  # empty batch
    hostbuf = np.zeros(4 * 2 * 3 * 4, np.uint32)
    assert L.convgpu_wrap_ops(hostbuf.ctypes.data, 4, 3, 2, 512, out.data_ptr(), s) < 0


def test_wrap_full_size_sampled(orc):
    """Config-[2]-sized stream (10^6 traces x 64 x 4 records, 4 GB) through
    the bench launch configuration; 4,096 random columns checked against the
    oracle."""
    import torch

    import paper_conf_cluster_kangjkkk17_b200 as cg
    N, K, n = 1_000_000, 4, 64
    tile = W.random_api_batch(41, 256, n, K, "mixed")
    api = _dev(tile).repeat(N // 256, 1, 1, 1)
    out = cg.wrap_ops(api, n, K)
    torch.cuda.synchronize()
    rng = np.random.default_rng(42)
    idx = rng.integers(0, N, 4096)
    got = out[torch.from_numpy(idx).cuda()].cpu().numpy().view(np.uint32)
    want = orc.wrap_batch(tile, 512)[idx % 256]
    assert np.array_equal(got, want)
