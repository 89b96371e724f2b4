"""ConVGPU scheduler-replay ORACLE — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
`--impl reference` leg may import this package.  It wraps the plain C oracle
(oracle/oracle.c, built into oracle/liboracle.so with gcc) through ctypes and
ships an independent pure-Python brute-force explorer (oracle/bruteforce.py).
It never imports the product package and the product never imports it.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = [os.path.join(_HERE, "oracle.c"), os.path.join(_HERE, "wrapper.c")]

POLICY = {"fifo": 0, "best_fit": 1, "recent_fit": 2, "random_fit": 3}
NONE32 = 0xFFFFFFFF
NONE8 = 0xFF
FLAG_BITS = ("deadlock", "overcommit", "invalid_limit", "invalid_free",
             "unsorted_arrival", "tick_range", "bad_program")


def build(force: bool = False) -> str:
    """Compile the C oracle with gcc (plain -O2, no special tuning)."""
    newest = max(os.path.getmtime(p) for p in _SRC + [os.path.join(_HERE, "oracle.h")])
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < newest:
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-fPIC", "-shared",
                               "-o", _SO] + _SRC)
        exe = os.path.join(_HERE, "oracle_run")
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-o", exe,
                               os.path.join(_HERE, "oracle_run.c")] + _SRC)
    return _SO


class _Trace(C.Structure):
    _fields_ = [("n", C.c_uint32), ("K", C.c_uint32),
                ("arrival", C.POINTER(C.c_uint32)), ("limit", C.POINTER(C.c_uint32)),
                ("delta", C.POINTER(C.c_uint32)), ("arg", C.POINTER(C.c_uint32))]


class _Result(C.Structure):
    _fields_ = [("admit_tick", C.c_uint32 * 64), ("admit_rank", C.c_uint32 * 64),
                ("wait", C.c_uint32 * 64), ("finish", C.c_uint32 * 64),
                ("makespan", C.c_uint32), ("peak_reserved", C.c_uint32),
                ("peak_used", C.c_uint32), ("flags", C.c_uint32),
                ("sum_wait", C.c_uint64), ("n_rejected", C.c_uint32),
                ("n_select", C.c_uint32), ("digest", C.c_uint64),
                ("events", C.c_uint64), ("violation", C.c_int32),
                ("violation_event", C.c_uint64)]


class Stats(C.Structure):
    _fields_ = [("traces", C.c_uint64), ("events", C.c_uint64),
                ("sum_makespan", C.c_uint64), ("sum_wait", C.c_uint64),
                ("n_rejected", C.c_uint64), ("n_select", C.c_uint64),
                ("digest_sum", C.c_uint64), ("max_makespan", C.c_uint32),
                ("max_peak_reserved", C.c_uint32), ("flag_count", C.c_uint32 * 8)]

    def as_dict(self) -> dict:
        d = {f: getattr(self, f) for f, _ in self._fields_ if f != "flag_count"}
        d["flag_count"] = list(self.flag_count)
        return d


class _Gen(C.Structure):
    _fields_ = [("gen_seed", C.c_uint64), ("n", C.c_uint32), ("K", C.c_uint32),
                ("n_classes", C.c_uint32), ("class_mib", C.c_uint32 * 8),
                ("num", C.c_uint32), ("den", C.c_uint32), ("iat", C.c_uint32),
                ("dur_base", C.c_uint32), ("dur_step", C.c_uint32),
                ("dur_class_offset", C.c_uint32), ("dur_jit", C.c_uint32),
                ("ovh", C.c_uint32)]


class ApiOp(C.Structure):
    _fields_ = [("api", C.c_uint32), ("a0", C.c_uint32), ("a1", C.c_uint32), ("a2", C.c_uint32)]


API = {"malloc": 0, "malloc_managed": 1, "malloc_pitch": 2, "malloc_3d": 3, "free": 4,
       "mem_get_info": 5, "compute": 6, "exit": 7}
API_DTYPE = np.dtype([("api", np.uint32), ("a0", np.uint32), ("a1", np.uint32), ("a2", np.uint32)])

_lib = None


def build_fault(fault: int, out_dir: str) -> str:
    """TEST-ONLY: compile the oracle with -DORC_FAULT=<fault> (one planted bug,
    see oracle.c) into out_dir, so tests can show the invariant checker fires."""
    so = os.path.join(out_dir, f"liboracle_fault{fault}.so")
    subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-fPIC", "-shared",
                           f"-DORC_FAULT={int(fault)}", "-o", so] + _SRC)
    return so


def load(path: str):
    """ctypes handle with the oracle's prototypes declared (lib() or a fault build)."""
    return _declare(C.CDLL(path))


def lib():
    global _lib
    if _lib is None:
        build()
        _lib = _declare(C.CDLL(_SO))
    return _lib


def _declare(L):
    u32p, u64p, u8p = C.POINTER(C.c_uint32), C.POINTER(C.c_uint64), C.POINTER(C.c_uint8)
    L.orc_philox4x32_10.argtypes = [u32p, u32p, u32p]
    L.orc_mix64.argtypes = [C.c_uint64]
    L.orc_mix64.restype = C.c_uint64
    L.orc_replay.argtypes = [C.POINTER(_Trace), C.c_uint32, C.c_int, C.c_uint64,
                             C.c_uint64, C.c_uint32, C.c_int, C.POINTER(_Result)]
    L.orc_generate.argtypes = [C.POINTER(_Gen), C.c_uint64, u32p, u32p, u32p, u32p]
    L.orc_replay_range.argtypes = [C.POINTER(_Gen), C.c_uint32, C.c_int, C.c_uint64,
                                   C.c_uint32, C.c_uint64, C.c_uint64, C.c_int,
                                   C.POINTER(Stats), u32p, u64p, u32p, u32p, u8p,
                                   u32p, u32p]
    L.orc_replay_batch.argtypes = [C.c_uint32, C.c_uint32, C.c_uint64, u32p, u32p,
                                   u32p, u32p, C.c_uint32, C.c_int, C.c_uint64,
                                   C.c_uint64, C.c_uint32, C.c_int, C.POINTER(Stats),
                                   u32p, u64p, u32p, u32p, u8p, u32p, u32p]
    L.orc_wrap_bytes.argtypes = [C.POINTER(ApiOp), C.c_uint32]
    L.orc_wrap_bytes.restype = C.c_uint64
    L.orc_wrap_mib.argtypes = [C.c_uint64]
    L.orc_wrap_mib.restype = C.c_uint32
    L.orc_wrap_program.argtypes = [C.POINTER(ApiOp), C.c_uint32, C.c_uint32, u32p]
    L.orc_wrap_batch.argtypes = [C.c_uint32, C.c_uint32, C.c_uint64, C.c_void_p, C.c_uint32, u32p]
    return L


def _p(a, ct=C.c_uint32):
    return None if a is None else a.ctypes.data_as(C.POINTER(ct))


LITERAL = 0x100  # OR into the policy: literal re-select-on-every-release reading


def _pol(policy) -> int:
    return POLICY[policy] if isinstance(policy, str) else int(policy)


def philox4x32_10(ctr, key):
    c = np.ascontiguousarray(ctr, np.uint32)
    k = np.ascontiguousarray(key, np.uint32)
    out = np.zeros(4, np.uint32)
    lib().orc_philox4x32_10(_p(c), _p(k), _p(out))
    return [int(x) for x in out]


def mix64(z: int) -> int:
    return int(lib().orc_mix64(z & 0xFFFFFFFFFFFFFFFF))


def replay_trace(arrival, limit, delta, arg, cap, policy, tid=0, seed=0, ovh=0,
                 check=True) -> dict:
    """Replay one trace.  delta/arg are [K][n]."""
    arrival = np.ascontiguousarray(arrival, np.uint32)
    limit = np.ascontiguousarray(limit, np.uint32)
    delta = np.ascontiguousarray(delta, np.uint32)
    arg = np.ascontiguousarray(arg, np.uint32)
    n = arrival.shape[0]
    K = delta.shape[0]
    tr = _Trace(n, K, _p(arrival), _p(limit), _p(delta), _p(arg))
    res = _Result()
    rc = lib().orc_replay(C.byref(tr), cap, _pol(policy), tid, seed, ovh,
                          1 if check else 0, C.byref(res))
    if rc:
        raise ValueError(f"orc_replay rc={rc}")
    out = {f: getattr(res, f) for f, _ in _Result._fields_}
    for f in ("admit_tick", "admit_rank", "wait", "finish"):
        out[f] = list(out[f])[:n]
    return out


def gen_struct(g) -> _Gen:
    cm = (C.c_uint32 * 8)(*list(g.class_mib) + [0] * (8 - len(g.class_mib)))
    return _Gen(g.gen_seed, g.n, g.K, len(g.class_mib), cm, g.num, g.den, g.iat,
                g.dur_base, g.dur_step, g.dur_class_offset, g.dur_jit, g.ovh)


def generate(g, tid: int):
    n, K = g.n, g.K
    arrival = np.zeros(n, np.uint32); limit = np.zeros(n, np.uint32)
    delta = np.zeros((K, n), np.uint32); arg = np.zeros((K, n), np.uint32)
    rc = lib().orc_generate(C.byref(gen_struct(g)), tid, _p(arrival), _p(limit),
                            _p(delta), _p(arg))
    if rc:
        raise ValueError("orc_generate rc=%d" % rc)
    return arrival, limit, delta, arg


def generate_batch(g, tid_lo: int, count: int):
    """Oracle-side generation of a batch in the C-ABI layout ([N,n], [N,K,n])."""
    n, K = g.n, g.K
    A = np.zeros((count, n), np.uint32); Lm = np.zeros((count, n), np.uint32)
    D = np.zeros((count, K, n), np.uint32); R = np.zeros((count, K, n), np.uint32)
    gs = gen_struct(g)
    for i in range(count):
        rc = lib().orc_generate(C.byref(gs), tid_lo + i, _p(A[i]), _p(Lm[i]), _p(D[i]), _p(R[i]))
        if rc:
            raise ValueError("orc_generate rc=%d" % rc)
    return A, Lm, D, R


def _outputs(count, n, full):
    o = dict(sum_u32x4=np.zeros((count, 4), np.uint32), sum_u64x2=np.zeros((count, 2), np.uint64),
             cnt_u32x2=np.zeros((count, 2), np.uint32))
    if full:
        o.update(admit_tick=np.zeros((count, n), np.uint32),
                 admit_rank=np.zeros((count, n), np.uint8),
                 wait=np.zeros((count, n), np.uint32), finish=np.zeros((count, n), np.uint32))
    else:
        o.update(admit_tick=None, admit_rank=None, wait=None, finish=None)
    return o


def _pack(o, st):
    s = o["sum_u32x4"]; w = o["sum_u64x2"]; cnt = o["cnt_u32x2"]
    res = dict(stats=st.as_dict(), makespan=s[:, 0], peak_reserved=s[:, 1],
               peak_used=s[:, 2], flags=s[:, 3], sum_wait=w[:, 0], digest=w[:, 1],
               n_rejected=cnt[:, 0], n_select=cnt[:, 1])
    for f in ("admit_tick", "admit_rank", "wait", "finish"):
        if o[f] is not None:
            res[f] = o[f]
    return res


def replay_range(w, policy, tid_lo: int, tid_hi: int, full: bool = False,
                 check: bool = False, rand_seed=None, L=None):
    """Generate + replay global trace ids [tid_lo, tid_hi) of workload w
    (L: another oracle build from load(), e.g. a fault build; default lib())."""
    g = w.gen
    count = tid_hi - tid_lo
    o = _outputs(count, g.n, full)
    st = Stats()
    seed = w.rand_seed if rand_seed is None else rand_seed
    rc = (L or lib()).orc_replay_range(C.byref(gen_struct(g)), w.cap, _pol(policy), seed, w.ovh,
                                tid_lo, tid_hi, 1 if check else 0, C.byref(st),
                                _p(o["sum_u32x4"]), _p(o["sum_u64x2"], C.c_uint64),
                                _p(o["cnt_u32x2"]), _p(o["admit_tick"]),
                                _p(o["admit_rank"], C.c_uint8), _p(o["wait"]), _p(o["finish"]))
    res = _pack(o, st)
    res["rc"] = rc
    return res


def replay_batch(b, cap, policy, tid_base=0, rand_seed=0, ovh=0, check=False, full=True, L=None):
    """Replay a workloads.Batch (numpy) with the oracle (L: see replay_range)."""
    count, n, K = b.count, b.n, b.K
    o = _outputs(count, n, full)
    st = Stats()
    arrs = [np.ascontiguousarray(x, np.uint32) for x in (b.arrival, b.limit, b.delta, b.arg)]
    rc = (L or lib()).orc_replay_batch(n, K, count, *[_p(x) for x in arrs], cap, _pol(policy),
                                tid_base, rand_seed, ovh, 1 if check else 0, C.byref(st),
                                _p(o["sum_u32x4"]), _p(o["sum_u64x2"], C.c_uint64),
                                _p(o["cnt_u32x2"]), _p(o["admit_tick"]),
                                _p(o["admit_rank"], C.c_uint8), _p(o["wait"]), _p(o["finish"]))
    res = _pack(o, st)
    res["rc"] = rc
    return res


# ---- NEXT-3: wrapper-side size semantics (oracle/wrapper.c) ----
def wrap_bytes(api, a0=0, a1=0, a2=0, pitch_align=512) -> int:
    op = ApiOp(API[api] if isinstance(api, str) else api, a0, a1, a2)
    return int(lib().orc_wrap_bytes(C.byref(op), pitch_align))


def wrap_mib(nbytes: int) -> int:
    return int(lib().orc_wrap_mib(nbytes))


def wrap_program(ops, pitch_align=512):
    """ops: list of (api, a0, a1, a2) for one container -> list of op words."""
    K = len(ops)
    arr = (ApiOp * K)(*[ApiOp(API[o[0]] if isinstance(o[0], str) else o[0], *o[1:]) for o in ops])
    out = np.zeros(K, np.uint32)
    lib().orc_wrap_program(arr, K, pitch_align, _p(out))
    return [int(x) for x in out]


def wrap_batch(api, pitch_align=512):
    """api: structured array API_DTYPE [count, K, n] -> op_arg uint32 [count, K, n]."""
    api = np.ascontiguousarray(api, API_DTYPE)
    count, K, n = api.shape
    out = np.zeros((count, K, n), np.uint32)
    lib().orc_wrap_batch(n, K, count, api.ctypes.data, pitch_align, _p(out))
    return out
