"""NEXT-3 oracle pins: the wrapper module's size semantics (oracle/wrapper.c,
PAPER.md P:104-110, Table II; R13').

Pinned to things other than the oracle's own formula:
* the CUDA runtime on a B200 (tests/golden/b200_pitch_probe.json): the pitch
  cudaMallocPitch / cudaMalloc3D really return for ~2,000 row widths;
* the defining properties of "a multiple of 128 MiB" and of a MiB
  count that covers a byte count (least such multiple / count);
* the replay oracle and its invariant checker: a wrapped program that frees
  what it allocated never frees more than it holds; a double free, a free of
  a non-allocation and an unknown API code are flagged by the replay.
"""
import json
import os

import numpy as np
import pytest

import workloads as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
MIB = 1 << 20
ALLOC, FREE, FINISH, NOP = 0, 1, 2, 3


@pytest.fixture(scope="module")
def probe():
    with open(os.path.join(ROOT, "tests", "golden", "b200_pitch_probe.json")) as f:
        return json.load(f)


def test_pitch_matches_the_b200_runtime(orc, probe):
    A = probe["textureAlignment"]
    assert A == 512
    for w, pitch in probe["pitch"]:
        # height 1: the bytes the wrapper charges are exactly one pitched row
        assert orc.wrap_bytes("malloc_pitch", w, 1, pitch_align=A) == pitch, w
        assert orc.wrap_bytes("malloc_pitch", w, 3, pitch_align=A) == 3 * pitch, w
    for w, h, d, pitch in probe["pitch3d"]:
        assert orc.wrap_bytes("malloc_3d", w, h, d, pitch_align=A) == pitch * h * d


def test_managed_is_the_least_multiple_of_128_mib(orc):
    rng = np.random.default_rng(5)
    vals = [0, 1, 128 * MIB - 1, 128 * MIB, 128 * MIB + 1, (1 << 40) + 3] + \
           [int(x) for x in rng.integers(0, 1 << 44, 2000)]
    for b in vals:
        m = orc.wrap_bytes("malloc_managed", b & 0xFFFFFFFF, b >> 32)
        assert m % (128 * MIB) == 0 and m >= b and m - b < 128 * MIB, b
        assert orc.wrap_bytes("malloc", b & 0xFFFFFFFF, b >> 32) == b  # cudaMalloc: as asked


def test_mib_is_the_least_covering_count_and_saturates(orc):
    rng = np.random.default_rng(6)
    for b in [0, 1, MIB - 1, MIB, MIB + 1] + [int(x) for x in rng.integers(0, 1 << 50, 2000)]:
        m = orc.wrap_mib(b)
        assert m * MIB >= b and (m == 0 or (m - 1) * MIB < b), b
    assert orc.wrap_mib((1 << 30) * MIB) == (1 << 30) - 1
    assert orc.wrap_mib((1 << 64) - 1) == (1 << 30) - 1
    # a 3D extent whose product overflows 64 bits saturates (over-limit request)
    w = orc.wrap_program([("malloc_3d", 0xFFFFFFFF, 0xFFFFFFFF, 0xFFFFFFFF), ("exit", 0, 0, 0)])
    assert w[0] == (ALLOC << 30) | ((1 << 30) - 1)


def test_api_classes_map_to_scheduler_ops(orc):
    w = orc.wrap_program([("malloc", 5 * MIB, 0, 0), ("mem_get_info", 0, 0, 0),
                          ("compute", 0, 0, 0), ("free", 0, 0, 0), ("exit", 0, 0, 0)])
    assert [x >> 30 for x in w] == [ALLOC, NOP, NOP, FREE, FINISH]
    assert w[0] & 0x3FFFFFFF == 5 and w[3] & 0x3FFFFFFF == 5  # the hash of address -> size


def _replay(orc, arg, limit=1 << 20, cap=1 << 21):
    K, n = arg.shape
    arrival = np.arange(n, dtype=np.uint32)
    lim = np.full(n, limit, np.uint32)
    delta = np.ones((K, n), np.uint32)
    return orc.replay_trace(arrival, lim, delta, arg, cap, "fifo")


def test_wrapped_valid_programs_never_free_more_than_held(orc):
    api = W.random_api_batch(11, 40, 6, 6, "valid", scale_mib=512)
    words = orc.wrap_batch(api, 512)
    for i in range(api.shape[0]):
        r = _replay(orc, words[i])
        assert r["violation"] == 0
        assert not (r["flags"] & (1 << 3)), i  # INVALID_FREE
        assert not (r["flags"] & (1 << 6)), i  # BAD_PROGRAM


def test_bad_references_are_flagged_by_the_replay(orc):
    def one(prog):
        w = np.array(orc.wrap_program(prog), np.uint32).reshape(-1, 1)
        return _replay(orc, w)["flags"]
    ok = [("malloc", MIB, 0, 0), ("free", 0, 0, 0), ("exit", 0, 0, 0)]
    assert one(ok) == 0
    assert one([("malloc", MIB, 0, 0), ("free", 0, 0, 0), ("free", 0, 0, 0), ("exit", 0, 0, 0)]) & 8
    assert one([("mem_get_info", 0, 0, 0), ("free", 0, 0, 0), ("exit", 0, 0, 0)]) & 8
    assert one([("free", 1, 0, 0), ("malloc", MIB, 0, 0), ("exit", 0, 0, 0)]) & 8
    assert one([("malloc", MIB, 0, 0), (9, 0, 0, 0), ("exit", 0, 0, 0)]) & 64
    assert one([("malloc", MIB, 0, 0), ("compute", 0, 0, 0), (0xFFFFFFFF, 0, 0, 0)]) & 64


def test_mixed_batches_are_total(orc):
    """Every record of a hostile batch maps to a well-formed op word."""
    api = W.random_api_batch(12, 30, 7, 8, "mixed")
    words = orc.wrap_batch(api, 512)
    assert words.shape == api.shape
    kinds = words >> 30
    assert set(np.unique(kinds)) <= {ALLOC, FREE, FINISH, NOP}
