"""NEXT-4: the live scheduler daemon (convgpud, ctl/sched.cpp) driven
message by message through a trace must schedule exactly as the replay
oracle does: same admissions (tick, rank), suspended times, finish ticks,
rejections, selections and reserved peak, for every policy (CPU only; the
daemon never touches a GPU)."""
import numpy as np
import pytest

import workloads as W

from ctl_driver import drive

POLS = ["fifo", "best_fit", "recent_fit", "random_fit"]
KEYS = ["admit_tick", "admit_rank", "wait", "finish", "n_rejected", "n_select",
        "peak_reserved", "makespan", "flags"]


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_cluster_kangjkkk17_b200 import build
    build.build_ctl()


def _check(orc, tr, cap, pol, ovh=0, tid=0, seed=0):
    got = drive(tr, cap, pol, ovh=ovh, tid=tid, seed=seed)
    ref = orc.replay_trace(tr["arrival"], tr["limit"], tr["delta"], tr["arg"], cap, pol,
                           tid=tid, seed=seed, ovh=ovh)
    for k in KEYS:
        assert got[k] == ref[k], (pol, k, got[k], ref[k])
    return ref


@pytest.mark.parametrize("pol", POLS)
def test_fig3_live(orc, pol):
    f = W.fig3_fixture()
    ref = _check(orc, f, f["cap"], pol)
    assert ref["admit_tick"] == [0, 0, 50, 150]


@pytest.mark.parametrize("mode", ["valid", "delayed", "over"])
@pytest.mark.parametrize("pol", POLS)
def test_random_traces_live(orc, pol, mode):
    b = W.random_batch(21, 25, 6, 4, 24, mode=mode, max_arrival_step=2,
                       limit_choices=range(1, 25))
    sel = 0
    for i in range(b.count):
        tr = dict(arrival=b.arrival[i], limit=b.limit[i], delta=b.delta[i], arg=b.arg[i])
        ref = _check(orc, tr, 24, pol, tid=i, seed=5)
        sel += ref["n_select"]
    assert sel > 0  # the batch exercises the policy's selection


@pytest.mark.parametrize("pol", POLS)
def test_context_overhead_live(orc, pol):
    b = W.random_batch(22, 12, 5, 3, 30, ovh=2, mode="valid", max_arrival_step=1,
                       limit_choices=range(2, 31))
    for i in range(b.count):
        tr = dict(arrival=b.arrival[i], limit=b.limit[i], delta=b.delta[i], arg=b.arg[i])
        _check(orc, tr, 30, pol, ovh=2, tid=i, seed=1)


def _daemon(cap=100, pol="fifo", ovh=0):
    import os
    import tempfile

    from paper_conf_cluster_kangjkkk17_b200 import ctl
    path = os.path.join(tempfile.mkdtemp(prefix="cgd"), "s")
    return ctl, path, ctl.Daemon(path, cap, pol, ovh)


def test_protocol_edges():
    ctl, path, d = _daemon(100, ovh=6)
    with d:
        c = ctl.Client(path, pid=7)
        assert c.call(ctl.ALLOC, 5)[0] == ctl.PROTOCOL  # before HELLO
        assert c.call(ctl.HELLO, 40, 1)[:3] == (ctl.OK, ctl.HELLO, 0)
        assert c.call(ctl.HELLO, 40, 1)[0] == ctl.PROTOCOL  # twice
        assert c.call(ctl.MEMINFO)[2:4] == (40, 40)  # the container's own view
        assert c.call(ctl.ALLOC, 10)[0] == ctl.OK  # 10 + 6 context
        assert c.call(ctl.MEMINFO)[2:4] == (24, 40)
        assert c.call(ctl.ALLOC_DONE, 0xABC, 10)[0] == ctl.OK
        assert c.call(ctl.FREE, 0xDEF)[0] == ctl.INVALID  # unknown address
        assert c.call(ctl.FREE, 0xABC)[0] == ctl.OK  # its recorded size
        assert c.call(ctl.FREE, 0xABC)[0] == ctl.INVALID  # already freed
        assert c.call(ctl.MEMINFO)[2:4] == (34, 40)  # the context stays charged
        assert c.call(ctl.ALLOC, 35)[0] == ctl.REJECT  # 6 + 35 > 40
        assert c.call(ctl.FREE_BYTES, 7)[0] == ctl.INVALID  # more than it uses (R11)
        st = c.call(ctl.STATS)
        assert st[2] == 60 and st[4] == 1  # pool 100 - 40; one rejection
        assert c.call(99)[0] == ctl.PROTOCOL
        c.close()


def test_multi_process_container_and_disconnect():
    """Processes with the same key share one container; it finishes (and
    its memory returns to the pool) only when the last one is gone — by EXIT
    or by disconnecting."""
    ctl, path, d = _daemon(100, ovh=0)
    with d:
        cc = ctl.Client(path, pid=0)
        p1, p2 = ctl.Client(path, pid=1), ctl.Client(path, pid=2)
        assert p1.call(ctl.HELLO, 60, 5)[2] == 0
        assert p2.call(ctl.HELLO, 60, 5)[2] == 0  # joins container 0
        assert cc.call(ctl.STATS)[2] == 40
        other = ctl.Client(path, pid=3)
        assert other.call(ctl.HELLO, 50, 6)[2] == 1  # gets 40 of 50: fill target
        other.send(ctl.ALLOC, 45)  # paused: its reply is withheld
        assert p1.call(ctl.EXIT)[0] == ctl.OK
        assert other.recv(block=False) is None  # container 0 still has p2
        p2.close()  # p2 vanishes without EXIT
        rep = other.recv()  # resumed when container 0 finished (Fig. 3)
        assert rep[:2] == (ctl.OK, ctl.ALLOC)
        assert cc.call(ctl.INFO, 1)[2:5] == (50, 45, 1)  # admitted (rank 1), its full limit
        other.close()
        p1.close()
        cc.close()


def test_disconnect_while_paused_withdraws_the_request():
    """A process whose ALLOC paused its container disconnects while another
    process of the same container has an ALLOC queued: the dead request is
    withdrawn, and the queued one goes through its own admission check
    instead of inheriting the dead request's grant (so the container never
    uses more than its declared limit, P:7)."""
    ctl, path, d = _daemon(100, ovh=0)
    with d:
        cc = ctl.Client(path, pid=0)
        a = ctl.Client(path, pid=1)
        assert a.call(ctl.HELLO, 60, 1)[2] == 0  # admitted with 60
        b1, b2 = ctl.Client(path, pid=2), ctl.Client(path, pid=3)
        assert b1.call(ctl.HELLO, 50, 2)[2] == 1  # 40 of 50: fill target
        assert b2.call(ctl.HELLO, 50, 2)[2] == 1
        b1.send(ctl.ALLOC, 45)  # 45 > 40 assigned: paused
        b2.send(ctl.ALLOC, 40)  # queued behind b1's request
        cc.call(ctl.SYNC)
        assert b2.recv(block=False) is None
        b1.close()  # b1 dies with its request paused
        rep = b2.recv()  # b2's own request: 40 <= 40 assigned, granted
        assert rep[:2] == (ctl.OK, ctl.ALLOC)
        assert cc.call(ctl.INFO, 1)[2:4] == (40, 40)
        assert b2.call(ctl.ALLOC, 20)[0] == ctl.REJECT  # 60 > limit 50
        assert cc.call(ctl.INFO, 1)[2:4] == (40, 40)
        assert a.call(ctl.EXIT)[0] == ctl.OK  # A's 60 returns; B filled to 50
        assert cc.call(ctl.INFO, 1)[2:5] == (50, 40, 1)
        b2.close()
        a.close()
        assert cc.call(ctl.STATS)[2] == 100
        cc.close()


def test_alloc_after_exit_is_refused():
    """After EXIT the process's container has given its memory back: a later
    ALLOC / FREE from that connection is a protocol error and charges
    nothing, so the pool is whole again after the disconnect."""
    ctl, path, d = _daemon(100, ovh=0)
    with d:
        cc = ctl.Client(path, pid=0)
        p = ctl.Client(path, pid=1)
        assert p.call(ctl.HELLO, 60, 1)[0] == ctl.OK
        assert cc.call(ctl.STATS)[2] == 40
        assert p.call(ctl.EXIT)[0] == ctl.OK
        assert cc.call(ctl.STATS)[2] == 100
        assert p.call(ctl.ALLOC, 10)[0] == ctl.PROTOCOL
        assert p.call(ctl.FREE_BYTES, 1)[0] == ctl.PROTOCOL
        assert p.call(ctl.ALLOC_DONE, 0x10, 10)[0] == ctl.PROTOCOL
        p.close()
        assert cc.call(ctl.STATS)[2] == 100
        cc.close()
