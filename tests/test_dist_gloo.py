"""N>1 host logic on CPU: world_size-2 gloo process group.  Each rank takes
its contiguous trace-id shard, replays it (here with the oracle, since there
is no GPU), packs the result into the convgpu_stats_t record and reduces it
with paper_conf_cluster_kangjkkk17_b200.dist — the result must equal the
single-process replay of the whole range."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import workloads as W
from paper_conf_cluster_kangjkkk17_b200 import STATS_DTYPE
from paper_conf_cluster_kangjkkk17_b200 import dist as cgd

TOTAL = 3001
RANGE = 256


def _pack(st: dict) -> torch.Tensor:
    rec = np.zeros(1, STATS_DTYPE)
    for k, v in st.items():
        if k == "flag_count":
            rec[0][k] = v
        else:
            rec[0][k] = v & (2**64 - 1)
    return torch.from_numpy(rec.view(np.int64).copy())


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, policy, q):
    import torch.distributed as dist

    import oracle
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        w = W.CONFIGS["c1"]
        lo, hi = cgd.shard_range(TOTAL, rank, world)
        r = oracle.replay_range(w, policy, lo, hi)
        st = _pack(r["stats"])
        blk = torch.stack([st, st]).contiguous()  # the batched form: two records at once
        cgd.reduce_stats(st)
        cgd.reduce_stats_block(blk)
        assert (blk[0] == st).all() and (blk[1] == st).all()
        rdu = np.zeros((TOTAL + RANGE - 1) // RANGE, np.uint64)
        with np.errstate(over="ignore"):
            np.add.at(rdu, (lo + np.arange(hi - lo)) // RANGE, r["digest"].astype(np.uint64))
        rd = torch.from_numpy(rdu.view(np.int64))
        cgd.reduce_range_digests(rd)
        m = cgd.max_over_ranks(float(rank + 1), torch.device("cpu"))
        q.put((rank, st.numpy().copy(), rd.numpy().copy(), m))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("policy", ["best_fit", "random_fit"])
def test_two_rank_stats_reduce_equals_single_process(orc, policy):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, policy, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    full = orc.replay_range(W.CONFIGS["c1"], policy, 0, TOTAL)
    want = _pack(full["stats"]).numpy()
    for rank, st, rd, m in res:
        np.testing.assert_array_equal(st, want)
        assert m == 2.0
        exp = np.zeros(len(rd), np.uint64)
        with np.errstate(over="ignore"):
            np.add.at(exp, np.arange(TOTAL) // RANGE, full["digest"].astype(np.uint64))
        np.testing.assert_array_equal(rd.view(np.uint64), exp)


def test_shard_range_partitions():
    for total in (0, 1, 7, 10**8 + 3):
        for world in (1, 2, 3, 8):
            spans = [cgd.shard_range(total, r, world) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == total
            assert all(a[1] == b[0] for a, b in zip(spans, spans[1:]))
            assert max(h - l for l, h in spans) - min(h - l for l, h in spans) <= 1
    with pytest.raises(ValueError):
        cgd.shard_range(10, 2, 2)


def test_reduce_stats_single_process_is_identity():
    t = torch.arange(12, dtype=torch.int64)
    assert (cgd.reduce_stats(t.clone()) == t).all()
    with pytest.raises(ValueError):
        cgd.reduce_stats(torch.zeros(11, dtype=torch.int64))
