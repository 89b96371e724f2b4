"""Drive a live convgpud with a replay trace (NEXT-4 parity, test
infrastructure).

The driver is a discrete-event loop over the trace in the replay's total
order (tick, container) (R16): an arrival is a container's HELLO, an op is
an ALLOC / FREE_BYTES / EXIT message on that container's connection, a NOP
sends nothing.  An ALLOC whose reply is withheld (found silent after a SYNC
barrier) pauses the container; every later step's withheld replies resume
containers at that step's tick, and the container's next op then runs at
resume tick + delta (R17).  After each event the driver reads admissions
(INFO) and the reserved peak (STATS).  It returns the fields the oracle's
replay returns for the same trace.
"""
import os
import tempfile

from paper_conf_cluster_kangjkkk17_b200 import ctl

NONE32 = 0xFFFFFFFF
SIZE = 0x3FFFFFFF


def drive(tr, cap, policy, ovh=0, tid=0, seed=0):
    arrival, limit, delta, arg = tr["arrival"], tr["limit"], tr["delta"], tr["arg"]
    n, K = len(arrival), len(delta)
    path = os.path.join(tempfile.mkdtemp(prefix="cgd"), "s")
    out = dict(admit_tick=[NONE32] * n, admit_rank=[0xFF] * n, wait=[0] * n, finish=[0] * n,
               n_rejected=0, peak_reserved=0, flags=0)
    with ctl.Daemon(path, cap, policy, ovh, seed=seed, tid=tid):
        cc = ctl.Client(path, pid=0)
        sent = [0]

        def send(cl, typ, a=0, b=0):
            cl.send(typ, a, b)
            sent[0] += 1

        def call(cl, typ, a=0, b=0):
            send(cl, typ, a, b)
            return cl.recv()

        def barrier():  # every message sent so far has been handled
            while True:
                before = sent[0]
                rep = call(cc, ctl.SYNC)
                if rep[2] >= before:
                    return

        conn = [None] * n
        k = [0] * n
        nxt = [0] * n
        state = ["pending"] * n  # pending / live / paused / done
        susp = [0] * n

        def advance(c, t):
            k[c] += 1
            nxt[c] = t + int(delta[k[c]][c])

        while True:
            cand = [(int(arrival[c]), c) for c in range(n) if state[c] == "pending"] + \
                   [(nxt[c], c) for c in range(n) if state[c] == "live"]
            if not cand:
                if any(s == "paused" for s in state):
                    out["flags"] |= 1  # DEADLOCK
                break
            t, c = min(cand)
            if state[c] == "pending":
                conn[c] = ctl.Client(path, pid=c + 1)
                rep = call(conn[c], ctl.HELLO, int(limit[c]), c)
                assert rep[0] == ctl.OK and rep[2] == c
                state[c] = "live"
                nxt[c] = t + int(delta[0][c])
            else:
                w = int(arg[k[c]][c])
                kind, r = w >> 30, w & SIZE
                if kind == 0:  # ALLOC
                    send(conn[c], ctl.ALLOC, r)
                    barrier()
                    rep = conn[c].recv(block=False)
                    if rep is None:
                        state[c] = "paused"
                        susp[c] = t
                    else:
                        if rep[0] == ctl.REJECT:
                            out["n_rejected"] += 1
                        advance(c, t)
                elif kind == 1:  # FREE
                    rep = call(conn[c], ctl.FREE_BYTES, r)
                    if rep[0] != ctl.OK:
                        out["flags"] |= 8  # INVALID_FREE
                        break
                    advance(c, t)
                elif kind == 3:  # NOP
                    advance(c, t)
                else:  # FINISH
                    rep = call(conn[c], ctl.EXIT)
                    assert rep[0] == ctl.OK
                    state[c] = "done"
                    out["finish"][c] = t
            # withheld replies released by this step: the containers resume at t
            for p in range(n):
                if state[p] == "paused":
                    rep = conn[p].recv(block=False)
                    if rep is not None:
                        assert rep[0] == ctl.OK
                        out["wait"][p] += t - susp[p]
                        state[p] = "live"
                        advance(p, t)
            for p in range(n):
                if state[p] != "pending" and out["admit_tick"][p] == NONE32:
                    rep = call(cc, ctl.INFO, p)
                    if rep[4] != ctl.NONE64:
                        out["admit_tick"][p] = t
                        out["admit_rank"][p] = rep[4]
            st = call(cc, ctl.STATS)
            out["peak_reserved"] = max(out["peak_reserved"], cap - st[2])
        st = call(cc, ctl.STATS)
        out["n_select"] = st[3]
        for cl in conn:
            if cl is not None:
                cl.close()
        cc.close()
    out["makespan"] = max(out["finish"]) - int(arrival[0]) if not out["flags"] else 0
    return out
