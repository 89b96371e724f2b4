"""Seeded synthetic workload recipes shared by the oracle and the CUDA path.

This module holds NO scheduler arithmetic: it only names the workload
parameters of BASELINE.json's configs (DESIGN.md §Input recipe), the Fig. 3
fixture inputs (numbers chosen in DESIGN.md R-Fig3) and
numpy builders of small seeded edge-case traces.  Both `oracle/` and the
product package receive their inputs from here; neither imports the other.

Trace layout (the C-ABI batch layout, include/convgpu.h):
  arrival[i][c], limit[i][c]          uint32, MiB / ticks
  op_delta[i][k][c], op_arg[i][k][c]  uint32; op_arg = kind << 30 | size_mib
"""
from __future__ import annotations

import dataclasses
from dataclasses import dataclass, field

import numpy as np

ALLOC, FREE, FINISH, NOP = 0, 1, 2, 3
POLICIES = ("fifo", "best_fit", "recent_fit", "random_fit")
# Table III GPU memory column, P:181-187 (MiB).
TABLE_III_MIB = (128, 256, 512, 1024, 2048, 4096)


def op(kind: int, size: int = 0) -> int:
    """Encode one op word (input format only)."""
    return (kind << 30) | size


@dataclass(frozen=True)
class GenParams:
    """Counter-based generator parameters; field-for-field the C structs."""
    gen_seed: int = 0x00C0FFEE
    n: int = 64
    K: int = 4
    class_mib: tuple = TABLE_III_MIB
    num: int = 1
    den: int = 1
    iat: int = 5000
    dur_base: int = 5000
    dur_step: int = 8000
    dur_class_offset: int = 0
    dur_jit: int = 0
    ovh: int = 0


@dataclass(frozen=True)
class Workload:
    name: str
    gen: GenParams
    cap: int                 # GPU capacity, MiB
    n_traces: int
    ovh: int = 0             # replay-side per-process context overhead
    rand_seed: int = 0       # Random-Fit key
    note: str = ""

    def events_per_trace(self) -> int:
        return self.gen.n * (1 + self.gen.K)


# BASELINE.json configs (0-based), DESIGN.md §Input recipe.
CONFIGS = {
    "c1": Workload(
        "c1_1e4x16", GenParams(n=16, K=4, class_mib=(512, 1024, 2048, 4096),
                               num=1, den=1, iat=5000, dur_class_offset=2),
        cap=8192, n_traces=10_000,
        note="10^4 traces x 16 containers, 0.5-4 GiB limits, 8 GiB GPU"),
    "c2": Workload(
        "c2_1e6x64_rho2", GenParams(n=64, K=4, class_mib=TABLE_III_MIB,
                                    num=30, den=7, iat=100),
        cap=184_320, n_traces=1_000_000,
        note="10^6 traces x 64 containers, 2x oversubscription of 180 GiB"),
    "c3": Workload(
        "c3_1e8x64_rho2", GenParams(n=64, K=4, class_mib=TABLE_III_MIB,
                                    num=30, den=7, iat=100),
        cap=184_320, n_traces=100_000_000,
        note="config [2] generator, 10^8 traces sharded over ranks"),
    # NEXT-2: paper-mimic (P:175 5 GB K20m, P:179 one container every 5 s,
    # ALLOC L-66 then run 5-45 s, P:135 66 MiB context).
    "mimic": Workload(
        "paper_mimic", GenParams(n=38, K=2, class_mib=TABLE_III_MIB, num=1,
                                 den=1, iat=5000, ovh=66),
        cap=5120, n_traces=10_000, ovh=66),
}


def rho_sweep(rho: int, n_traces: int = 1_000_000, rand_seed: int = 0) -> Workload:
    """Config [4]: 180 GiB capacity, limits scaled by 15*rho/7 (E[sum L]/cap=rho)."""
    return Workload(f"c4_rho{rho}", GenParams(n=64, K=4, class_mib=TABLE_III_MIB,
                                              num=15 * rho, den=7, iat=100),
                    cap=184_320, n_traces=n_traces, rand_seed=rand_seed)


# ---------------------------------------------------------------------------
# Config [0]: the Fig. 3 fixture.  The paper gives the story, not
# numbers; DESIGN.md R-Fig3 picks these.  Expected outputs: tests/golden.
def fig3_fixture():
    arrival = np.array([0, 0, 10, 20], np.uint32)
    limit = np.array([3072, 3072, 4096, 3072], np.uint32)
    K = 3
    delta = np.zeros((K, 4), np.uint32)
    arg = np.zeros((K, 4), np.uint32)
    # A: ALLOC 3072 @0, FINISH @200 (NOP pads to K=3 before FINISH)
    # B: ALLOC 3072 @0, FINISH @50
    # C: ALLOC 1024 @0, ALLOC 2048 @10, FINISH @100
    # D: ALLOC 3072 @0, FINISH @100
    progs = [
        [(ALLOC, 3072, 0), (NOP, 0, 0), (FINISH, 0, 200)],
        [(ALLOC, 3072, 0), (NOP, 0, 0), (FINISH, 0, 50)],
        [(ALLOC, 1024, 0), (ALLOC, 2048, 10), (FINISH, 0, 100)],
        [(ALLOC, 3072, 0), (NOP, 0, 0), (FINISH, 0, 100)],
    ]
    for c, prog in enumerate(progs):
        for k, (kind, size, d) in enumerate(prog):
            delta[k, c] = d
            arg[k, c] = op(kind, size)
    return dict(arrival=arrival, limit=limit, delta=delta, arg=arg, cap=8192)


# ---------------------------------------------------------------------------
@dataclass
class Batch:
    """A batch of traces in the C-ABI layout (numpy, host)."""
    n: int
    K: int
    arrival: np.ndarray   # [N, n]
    limit: np.ndarray     # [N, n]
    delta: np.ndarray     # [N, K, n]
    arg: np.ndarray       # [N, K, n]

    @property
    def count(self) -> int:
        return self.arrival.shape[0]


def _program(rng, L, K, ovh, mode):
    """One container program of K ops ending in FINISH (input recipe only)."""
    kinds, sizes, deltas = [], [], []
    used = 0
    budget = max(L - ovh, 0)
    for k in range(K - 1):
        d = int(rng.integers(0, 4))
        if mode == "delayed" and k == 0:
            d = int(rng.integers(1, 6))
        r = rng.random()
        if r < 0.55:
            room = budget - used
            sz = int(rng.integers(0, room + 1)) if room > 0 else 0
            if mode == "over" and rng.random() < 0.3:
                sz = room + int(rng.integers(1, 3))   # rejected: over the limit
            else:
                used += sz
            kinds.append(ALLOC); sizes.append(sz)
        elif r < 0.8 and used > 0:
            sz = int(rng.integers(0, used + 1))
            if mode == "badfree" and rng.random() < 0.5:
                sz = used + 1
            kinds.append(FREE); sizes.append(sz)
            used -= min(sz, used)
        else:
            kinds.append(NOP); sizes.append(0)
        deltas.append(d)
    kinds.append(FINISH); sizes.append(0); deltas.append(int(rng.integers(0, 5)))
    return kinds, sizes, deltas


def random_batch(seed: int, count: int, n: int, K: int, cap: int, ovh: int = 0,
                 mode: str = "valid", max_arrival_step: int = 3,
                 limit_choices=None) -> Batch:
    """Seeded small random traces.  mode selects an edge-case mix:
    'valid' | 'delayed' (first op later than arrival) | 'over' (some ALLOCs
    over the limit) | 'badfree' (FREE > used) | 'unsorted' | 'biglimit'
    (L > cap) | 'badprog' (FINISH misplaced) | 'mixed' (all of the above)."""
    rng = np.random.default_rng(seed)
    arrival = np.zeros((count, n), np.uint32)
    limit = np.zeros((count, n), np.uint32)
    delta = np.zeros((count, K, n), np.uint32)
    arg = np.zeros((count, K, n), np.uint32)
    modes = ["valid", "delayed", "over", "badfree", "unsorted", "biglimit", "badprog"]
    for i in range(count):
        m = mode if mode != "mixed" else modes[int(rng.integers(0, len(modes)))]
        t = 0
        for c in range(n):
            t += int(rng.integers(0, max_arrival_step + 1))
            arrival[i, c] = t
            if limit_choices is not None:
                L = int(rng.choice(limit_choices))
            else:
                L = int(rng.integers(0, cap + 1))
            limit[i, c] = L
            kinds, sizes, deltas = _program(rng, L, K, ovh, m)
            for k in range(K):
                delta[i, k, c] = deltas[k]
                arg[i, k, c] = op(kinds[k], sizes[k])
        if m == "unsorted" and n > 1:
            c = int(rng.integers(1, n))
            arrival[i, c] = max(int(arrival[i, c - 1]) - 1, 0) if arrival[i, c - 1] > 0 else arrival[i, c]
            if arrival[i, c] >= arrival[i, c - 1]:
                arrival[i, c - 1] = arrival[i, c] + 1
        if m == "biglimit":
            limit[i, int(rng.integers(0, n))] = cap + 1
        if m == "badprog":
            c = int(rng.integers(0, n))
            k = int(rng.integers(0, K))
            if k == K - 1:
                arg[i, k, c] = op(NOP)
            else:
                arg[i, k, c] = op(FINISH)
    return Batch(n, K, arrival, limit, delta, arg)


def with_fields(w: Workload, **kw) -> Workload:
    return dataclasses.replace(w, **kw)


# ---------------------------------------------------------------------------
# NEXT-3: API-level programs (the wrapper module's input, PAPER.md P:104-110,
# Table II).  Records [count, K, n] of (api, a0, a1, a2) in the
# convgpu_api_op_t layout; API codes as in include/convgpu.h.  Input recipe
# only: random API calls and arguments, none of the size arithmetic.
API_MALLOC, API_MANAGED, API_PITCH, API_3D, API_FREE, API_MEMINFO, API_COMPUTE, API_EXIT = range(8)
API_RECORD = np.dtype([("api", np.uint32), ("a0", np.uint32), ("a1", np.uint32), ("a2", np.uint32)])


def _api_bytes(rng, scale_mib: int):
    """A byte count of log-uniform magnitude up to ~scale_mib MiB, as (lo, hi)."""
    top = max(int(scale_mib) << 20, 1)
    b = int(np.exp(rng.uniform(0.0, np.log(top + 1)))) - 1
    if rng.random() < 0.1:
        b = int(rng.choice([0, 1, (1 << 20) - 1, 1 << 20, (1 << 20) + 1, (128 << 20) - 1,
                            128 << 20, (128 << 20) + 1]))
    return b & 0xFFFFFFFF, b >> 32


def random_api_batch(seed: int, count: int, n: int, K: int, mode: str = "valid",
                     scale_mib: int = 4096) -> np.ndarray:
    """Seeded API-level programs.  'valid': allocations through the four
    allocation APIs, cudaFree of earlier allocations, cudaMemGetInfo /
    compute records, EXIT last.  'mixed': also frees naming later ops,
    non-allocations or freed allocations, unknown API codes anywhere, huge
    (saturating) arguments and a missing EXIT."""
    rng = np.random.default_rng(seed)
    out = np.zeros((count, K, n), API_RECORD)
    for i in range(count):
        for c in range(n):
            allocs = []
            for k in range(K):
                rec = [API_COMPUTE, 0, 0, 0]
                last = k == K - 1
                r = rng.random()
                if last and (mode == "valid" or rng.random() < 0.9):
                    rec = [API_EXIT, 0, 0, 0]
                elif r < 0.2:
                    lo, hi = _api_bytes(rng, scale_mib)
                    rec = [API_MALLOC, lo, hi, int(rng.integers(0, 1 << 32))]
                elif r < 0.35:
                    lo, hi = _api_bytes(rng, scale_mib)
                    rec = [API_MANAGED, lo, hi, 0]
                elif r < 0.6:
                    # moderate extents (<= 1 GiB); 'mixed' also draws full 32-bit ones
                    wide = mode != "valid"
                    big = lambda b: int(rng.integers(0, 1 << 32)) if wide and rng.random() < 0.2 \
                        else int(rng.integers(0, 1 << b))
                    if r < 0.5:
                        rec = [API_PITCH, big(16), big(14), int(rng.integers(0, 1 << 32))]
                    else:
                        rec = [API_3D, big(14), big(10), big(6)]
                elif r < 0.8:
                    live = [j for j in allocs]
                    if mode == "valid":
                        if live:
                            j = live[int(rng.integers(0, len(live)))]
                            allocs.remove(j)
                            rec = [API_FREE, j, 0, 0]
                        else:
                            rec = [API_MEMINFO, 0, 0, 0]
                    else:
                        rec = [API_FREE, int(rng.integers(0, K + 2)), 0, 0]
                elif r < 0.9:
                    rec = [API_MEMINFO, 0, 0, 0]
                if mode != "valid" and rng.random() < 0.05:
                    rec[0] = int(rng.choice([8, 9, 15, 0xFFFFFFFF]))
                if rec[0] <= API_3D and rec[0] < 8:
                    allocs.append(k)
                out[i, k, c] = tuple(rec)
    return out
