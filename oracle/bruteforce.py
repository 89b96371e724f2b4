"""Brute-force explorer of ConVGPU's scheduler — TEST INFRASTRUCTURE ONLY.

A third, independent implementation of the replay semantics (DESIGN.md
§Semantics), written in pure Python in a different style from oracle.c
(immutable-ish state copied at every branch, generator recursion).  Instead
of following one policy it EXPLORES, on tiny traces (config [0]):

  * every choice of fill target at every selection point ("there can
    exist multiple paused containers"; P:141-145 name four rules for the
    choice — the explorer tries all of them and any other), and
  * optionally every interleaving of same-tick events (the scheduler
    serialises steps with a mutex; the order of simultaneous requests is not
    fixed by the paper).

For every explored path it checks the paper's guarantees (P:7 "can prevent
the system from falling into deadlock"; P:91 consistency — memory in use
never exceeds capacity; P:149 every admitted container holds its declared
limit) and records which policy rules the path obeyed at every choice point,
so a test can compare "the path that obeys rule X in canonical event order"
with the C oracle's answer for policy X.
"""
from __future__ import annotations

import copy

MASK32 = 0xFFFFFFFF
ALLOC, FREE, FINISH, NOP = 0, 1, 2, 3


def philox4x32_10(ctr, key):
    """Philox4x32-10 (Salmon et al. SC'11), pure Python."""
    c = list(ctr)
    k0, k1 = key
    for r in range(10):
        if r:
            k0 = (k0 + 0x9E3779B9) & MASK32
            k1 = (k1 + 0xBB67AE85) & MASK32
        p0 = 0xD2511F53 * c[0]
        p1 = 0xCD9E8D57 * c[2]
        c = [((p1 >> 32) ^ c[1] ^ k0) & MASK32, p1 & MASK32,
             ((p0 >> 32) ^ c[3] ^ k1) & MASK32, p0 & MASK32]
    return c


class Violation(AssertionError):
    pass


class _S:
    """Scheduler state for one path."""

    def __init__(self, tr, cap, ovh, lit=False):
        n = len(tr["arrival"])
        self.lit = lit
        self.n = n
        self.cap = cap
        self.ovh = ovh
        self.free = cap
        self.target = None
        self.seq = 0
        self.rank = 0
        self.nsel = 0
        self.nrej = 0
        self.peak_res = 0
        self.peak_used = 0
        self.flags = 0
        self.stopped = False
        self.state = ["pending"] * n
        self.a = [0] * n
        self.used = [0] * n
        self.k = [0] * n
        self.nt = [0] * n
        self.paused = [False] * n
        self.pend = [0] * n
        self.stick = [0] * n
        self.sseq = [0] * n
        self.first = [False] * n
        self.admitted = [False] * n
        self.wait = [0] * n
        self.atick = [MASK32] * n
        self.arank = [0xFF] * n
        self.fin = [0] * n
        # policy conformance along this path
        self.obeys = {"fifo", "best_fit", "recent_fit", "random_fit"}
        self.canonical = True
        self.choices = []


def _checks(s, tr):
    L = tr["limit"]
    if sum(s.a) + s.free != s.cap:
        raise Violation("capacity ledger")
    if sum(s.used) > s.cap:
        raise Violation("memory in use exceeds capacity")
    if s.lit:  # the literal reading keeps partial holds: only the ledger checks apply
        for c in range(s.n):
            if not (0 <= s.used[c] <= s.a[c] <= L[c]):
                raise Violation("used <= a <= L")
        return
    partial = [c for c in range(s.n) if s.state[c] == "live" and 0 < s.a[c] < L[c]]
    if len(partial) > 1 or (partial and partial[0] != s.target):
        raise Violation("more than one partially assigned container")
    for c in range(s.n):
        if not (0 <= s.used[c] <= s.a[c] <= L[c]):
            raise Violation("used <= a <= L")
        if s.admitted[c] and s.state[c] == "live" and s.a[c] != L[c]:
            raise Violation("admitted container lost its guarantee")
    if s.target is not None and s.free != 0:
        raise Violation("target set but memory left unassigned")
    if s.target is None and any(s.paused):
        raise Violation("paused container with no fill target")


def _advance(s, tr, c, t):
    s.k[c] += 1
    K = len(tr["delta"])
    if s.k[c] < K:
        s.nt[c] = t + tr["delta"][s.k[c]][c]


def _admit(s, c, t):
    s.admitted[c] = True
    s.atick[c] = t
    s.arank[c] = s.rank
    s.rank += 1


def _apply(s, tr, c, t):
    L = tr["limit"][c]
    if s.state[c] == "pending":
        s.state[c] = "live"
        g = min(L, s.free) if (s.lit or s.target is None) else 0
        s.a[c] = g
        s.free -= g
        if g == L:
            _admit(s, c, t)
        elif g > 0 and not s.lit:
            s.target = c
        s.nt[c] = t + tr["delta"][0][c]
        return
    w = tr["arg"][s.k[c]][c]
    kind, size = w >> 30, w & 0x3FFFFFFF
    if kind == ALLOC:
        need = s.used[c] + size + (0 if s.first[c] else s.ovh)
        if need > L:
            s.nrej += 1
            _advance(s, tr, c, t)
        elif need <= s.a[c]:
            s.used[c] = need
            s.first[c] = True
            _advance(s, tr, c, t)
        else:
            s.paused[c] = True
            s.pend[c] = need - s.used[c]
            s.stick[c] = t
            s.sseq[c] = s.seq
            s.seq += 1
    elif kind == FREE:
        if size > s.used[c]:
            s.flags |= 1 << 3
            s.stopped = True
            return
        s.used[c] -= size
        _advance(s, tr, c, t)
    elif kind == FINISH:
        s.free += s.a[c]
        s.a[c] = 0
        s.used[c] = 0
        s.state[c] = "done"
        s.fin[c] = t
        if s.target == c:
            s.target = None
    else:
        _advance(s, tr, c, t)


def _rule_picks(s, tr, tid, seed):
    """What each named rule would pick right now (R3-R7)."""
    P = [c for c in range(s.n) if s.paused[c]]
    L = tr["limit"]
    picks = {}
    picks["fifo"] = min(P, key=lambda c: (tr["arrival"][c], c))
    need = {c: L[c] - s.a[c] for c in P}
    fit = [c for c in P if need[c] <= s.free]
    if fit:
        picks["best_fit"] = min(fit, key=lambda c: (s.free - need[c], c))
    else:
        picks["best_fit"] = min(P, key=lambda c: (need[c], c))
    picks["recent_fit"] = max(P, key=lambda c: s.sseq[c])
    x = philox4x32_10([tid & MASK32, tid >> 32, s.nsel & MASK32, 1],
                      [seed & MASK32, seed >> 32])
    picks["random_fit"] = sorted(P)[(x[0] * len(P)) >> 32]
    return P, picks


def _dispatch_lit(s, tr, t, tid, seed):
    """Literal reading (R1-LIT): while memory is free and someone is paused,
    ANY paused container may be chosen; it receives min(free, L - a)."""
    L = tr["limit"]
    if s.free == 0 or not any(s.paused):
        yield s
        return
    P, picks = _rule_picks(s, tr, tid, seed)
    for i, c in enumerate(P):
        s2 = copy.deepcopy(s) if i < len(P) - 1 else s
        s2.obeys = {p for p in s2.obeys if picks[p] == c}
        s2.choices.append(("select", c, tuple(P)))
        s2.nsel += 1
        g = min(s2.free, L[c] - s2.a[c])
        s2.a[c] += g
        s2.free -= g
        if s2.paused[c] and s2.used[c] + s2.pend[c] <= s2.a[c]:
            s2.used[c] += s2.pend[c]
            s2.first[c] = True
            s2.paused[c] = False
            s2.wait[c] += t - s2.stick[c]
            _advance(s2, tr, c, t)
        if s2.a[c] == L[c]:
            _admit(s2, c, t)
        yield from _dispatch_lit(s2, tr, t, tid, seed)


def _dispatch(s, tr, t, tid, seed):
    """Yield every state reachable by DISPATCH, branching on selections."""
    if s.lit:
        yield from _dispatch_lit(s, tr, t, tid, seed)
        return
    L = tr["limit"]
    while True:
        if s.target is not None:
            tg = s.target
            g = min(s.free, L[tg] - s.a[tg])
            s.a[tg] += g
            s.free -= g
            if s.paused[tg] and s.used[tg] + s.pend[tg] <= s.a[tg]:
                s.used[tg] += s.pend[tg]
                s.first[tg] = True
                s.paused[tg] = False
                s.wait[tg] += t - s.stick[tg]
                _advance(s, tr, tg, t)
            if s.a[tg] == L[tg]:
                _admit(s, tg, t)
                s.target = None
                continue
            yield s
            return
        if not any(s.paused):
            yield s
            return
        P, picks = _rule_picks(s, tr, tid, seed)
        for i, c in enumerate(P):
            s2 = copy.deepcopy(s) if i < len(P) - 1 else s
            s2.obeys = {p for p in s2.obeys if picks[p] == c}
            s2.choices.append(("select", c, tuple(P)))
            s2.target = c
            s2.nsel += 1
            yield from _dispatch(s2, tr, t, tid, seed)
        return


def _run(s, tr, tid, seed, permute_ties):
    while True:
        if s.stopped:
            yield s
            return
        cands = []
        for c in range(s.n):
            if s.state[c] == "pending":
                cands.append((tr["arrival"][c], c))
            elif s.state[c] == "live" and not s.paused[c]:
                cands.append((s.nt[c], c))
        if not cands:
            if any(st != "done" for st in s.state):
                s.flags |= 1
                if not s.lit:
                    raise Violation("deadlock: containers remain but none can run")
                s.stopped = True
            yield s
            return
        cands.sort()
        t0 = cands[0][0]
        options = [cands[0]] if not permute_ties else [x for x in cands if x[0] == t0]
        for i, (t, c) in enumerate(options):
            s2 = copy.deepcopy(s) if i < len(options) - 1 else s
            if i > 0:
                s2.canonical = False
            _apply(s2, tr, c, t)
            if s2.stopped:
                yield s2
                continue
            for s3 in list(_dispatch(s2, tr, t, tid, seed)):
                s3.peak_res = max(s3.peak_res, s3.cap - s3.free)
                s3.peak_used = max(s3.peak_used, sum(s3.used))
                _checks(s3, tr)
                yield from _run(s3, tr, tid, seed, permute_ties)
        return


def outcome(s, tr):
    stopped = s.flags & ~2
    n = s.n
    if stopped:
        return dict(admit_tick=[MASK32] * n, admit_rank=[0xFF] * n, wait=[0] * n,
                    finish=[0] * n, makespan=0, peak_reserved=0, peak_used=0,
                    sum_wait=0, n_rejected=0, n_select=0, flags=s.flags)
    return dict(admit_tick=list(s.atick), admit_rank=list(s.arank), wait=list(s.wait),
                finish=list(s.fin), makespan=max(s.fin) - tr["arrival"][0],
                peak_reserved=s.peak_res, peak_used=s.peak_used, sum_wait=sum(s.wait),
                n_rejected=s.nrej, n_select=s.nsel, flags=s.flags)


def explore(tr, cap, ovh=0, tid=0, seed=0, permute_ties=False, max_paths=200000, lit=False):
    """Return a list of (outcome, obeyed_policies, canonical, choices) per path.

    tr: dict(arrival=[n], limit=[n], delta=[K][n], arg=[K][n]) of Python ints.
    Raises Violation if any path breaks a guarantee (incl. deadlock).
    """
    tr = {k: [list(map(int, r)) for r in v] if k in ("delta", "arg") else list(map(int, v))
          for k, v in tr.items() if k in ("arrival", "limit", "delta", "arg")}
    paths = []
    for s in _run(_S(tr, cap, ovh, lit), tr, tid, seed, permute_ties):
        paths.append((outcome(s, tr), frozenset(s.obeys), s.canonical, tuple(s.choices)))
        if len(paths) > max_paths:
            raise RuntimeError("path explosion")
    return paths
