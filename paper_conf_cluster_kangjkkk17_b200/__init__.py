"""B200-native batched replay of ConVGPU's GPU-memory scheduler.

Thin Python binding over the C ABI of libconvgpu.so (include/convgpu.h):
argument marshalling only — every step of the replay (event loop, policy
selection, outputs, digests, statistics) and the synthetic generator run in
the sm_100a kernels.  PyTorch provides device memory and streams.  There is
no CPU fallback: if the extension is missing or the device is not sm_100 the
calls raise.

Paper: Kang et al., "ConVGPU", IEEE CLUSTER 2017.  Semantics and
readings: DESIGN.md.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass
from typing import Optional

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
# CONVGPU_SO: an alternative build of the same library (A/B kernel tuning only)
SO_PATH = os.environ.get("CONVGPU_SO") or os.path.join(_PKG, "libconvgpu.so")

FIFO, BEST_FIT, RECENT_FIT, RANDOM_FIT = 0, 1, 2, 3
LITERAL = 0x100  # CONVGPU_DISPATCH_LITERAL: OR into a policy for the R1-LIT reading
POLICY = {"fifo": FIFO, "best_fit": BEST_FIT, "recent_fit": RECENT_FIT, "random_fit": RANDOM_FIT}
ALLOC, FREE, FINISH, NOP = 0, 1, 2, 3
NONE32, NONE8 = 0xFFFFFFFF, 0xFF
KERNEL = {"auto": 0, "warp": 1, "lane": 2, "lane16": 3, "lane16w": 4}
FLAG_NAMES = ("deadlock", "overcommit", "invalid_limit", "invalid_free", "unsorted_arrival",
              "tick_range", "bad_program")

SUMMARY_DTYPE = np.dtype([("makespan", "<u4"), ("peak_reserved", "<u4"), ("peak_used", "<u4"),
                          ("flags", "<u4"), ("sum_wait", "<u8"), ("n_rejected", "<u4"),
                          ("n_select", "<u4"), ("digest", "<u8")])
STATS_DTYPE = np.dtype([("traces", "<u8"), ("events", "<u8"), ("sum_makespan", "<u8"),
                        ("sum_wait", "<u8"), ("n_rejected", "<u8"), ("n_select", "<u8"),
                        ("digest_sum", "<u8"), ("max_makespan", "<u4"),
                        ("max_peak_reserved", "<u4"), ("flag_count", "<u4", (8,))])
assert SUMMARY_DTYPE.itemsize == 40 and STATS_DTYPE.itemsize == 96


class ConvgpuError(RuntimeError):
    pass


# ---------------------------------------------------------------- ctypes ABI
class TracesT(C.Structure):
    _fields_ = [("arrival", C.c_void_p), ("limit", C.c_void_p), ("op_delta", C.c_void_p),
                ("op_arg", C.c_void_p), ("n_containers", C.c_uint32), ("n_ops", C.c_uint32),
                ("trace_id_base", C.c_uint64), ("rand_seed", C.c_uint64),
                ("ctx_overhead_mib", C.c_uint32), ("kernel_variant", C.c_uint32)]


class OutT(C.Structure):
    _fields_ = [("admit_tick", C.c_void_p), ("admit_rank", C.c_void_p), ("wait", C.c_void_p),
                ("finish", C.c_void_p), ("summary", C.c_void_p), ("stats", C.c_void_p),
                ("range_digest", C.c_void_p), ("range_size", C.c_uint64), ("stream", C.c_void_p),
                ("admit_scratch", C.c_void_p)]


class GenParamsT(C.Structure):
    _fields_ = [("gen_seed", C.c_uint64), ("n_containers", C.c_uint32), ("n_ops", C.c_uint32),
                ("n_classes", C.c_uint32), ("class_mib", C.c_uint32 * 8), ("num", C.c_uint32),
                ("den", C.c_uint32), ("iat", C.c_uint32), ("dur_base", C.c_uint32),
                ("dur_step", C.c_uint32), ("dur_class_offset", C.c_uint32),
                ("dur_jit", C.c_uint32), ("ctx_overhead_mib", C.c_uint32)]


class BuffersT(C.Structure):
    _fields_ = [("arrival", C.c_void_p), ("limit", C.c_void_p), ("op_delta", C.c_void_p),
                ("op_arg", C.c_void_p)]


class Traces16T(C.Structure):
    _fields_ = [("arrival", C.c_void_p), ("limit", C.c_void_p), ("op_size", C.c_void_p),
                ("op_delta", C.c_void_p), ("op_kinds", C.c_void_p),
                ("n_containers", C.c_uint32), ("n_ops", C.c_uint32),
                ("trace_id_base", C.c_uint64), ("rand_seed", C.c_uint64),
                ("ctx_overhead_mib", C.c_uint32), ("kernel_variant", C.c_uint32)]


class Buffers16T(C.Structure):
    _fields_ = [("arrival", C.c_void_p), ("limit", C.c_void_p), ("op_size", C.c_void_p),
                ("op_delta", C.c_void_p), ("op_kinds", C.c_void_p)]


EXPORTS = ("convgpu_replay", "convgpu_generate", "convgpu_replay_host",
           "convgpu_replay_host_workspace", "convgpu_wrap_ops", "convgpu_launches_per_call",
           "convgpu_strerror", "convgpu_abi_version", "convgpu_pack16", "convgpu_replay_host16",
           "convgpu_replay_host16_workspace")

# NEXT-3 API records (include/convgpu.h convgpu_api_t / convgpu_api_op_t)
API = {"malloc": 0, "malloc_managed": 1, "malloc_pitch": 2, "malloc_3d": 3, "free": 4,
       "mem_get_info": 5, "compute": 6, "exit": 7}
API_DTYPE = np.dtype([("api", np.uint32), ("a0", np.uint32), ("a1", np.uint32), ("a2", np.uint32)])
B200_PITCH_ALIGN = 512  # cudaDeviceProp.textureAlignment = cudaMallocPitch granule on B200

_lib = None


def lib():
    """Load the in-tree libconvgpu.so (built by __graft_entry__.build())."""
    global _lib
    if _lib is None:
        if not os.path.exists(SO_PATH):
            raise ConvgpuError(f"{SO_PATH} missing: run __graft_entry__.build() (no CPU fallback)")
        L = C.CDLL(SO_PATH)
        L.convgpu_replay.argtypes = [C.POINTER(TracesT), C.c_uint64, C.c_uint32, C.c_int,
                                     C.POINTER(OutT)]
        L.convgpu_generate.argtypes = [C.POINTER(GenParamsT), C.c_uint64, C.c_uint64,
                                       C.POINTER(BuffersT), C.c_void_p]
        L.convgpu_replay_host.argtypes = [C.POINTER(TracesT), C.c_uint64, C.c_uint32, C.c_uint32,
                                          C.c_void_p, C.c_void_p, C.c_void_p, C.c_size_t,
                                          C.c_uint64, C.c_void_p]
        L.convgpu_replay_host_workspace.argtypes = [C.c_uint32, C.c_uint32, C.c_uint64,
                                                    C.c_uint32]
        L.convgpu_replay_host_workspace.restype = C.c_size_t
        L.convgpu_wrap_ops.argtypes = [C.c_void_p, C.c_uint64, C.c_uint32, C.c_uint32, C.c_uint32,
                                       C.c_void_p, C.c_void_p]
        L.convgpu_pack16.argtypes = [C.POINTER(TracesT), C.c_uint64, C.POINTER(Buffers16T),
                                     C.c_void_p, C.c_void_p]
        L.convgpu_replay_host16.argtypes = [C.POINTER(Traces16T), C.c_uint64, C.c_uint32,
                                            C.c_uint32, C.c_void_p, C.c_void_p, C.c_void_p,
                                            C.c_size_t, C.c_uint64, C.c_void_p]
        L.convgpu_replay_host16_workspace.argtypes = [C.c_uint32, C.c_uint32, C.c_uint64,
                                                      C.c_uint32]
        L.convgpu_replay_host16_workspace.restype = C.c_size_t
        L.convgpu_strerror.argtypes = [C.c_int]
        L.convgpu_strerror.restype = C.c_char_p
        _lib = L
    return _lib


def _check(rc: int, what: str):
    if rc != 0:
        raise ConvgpuError(f"{what}: rc={rc} ({lib().convgpu_strerror(rc).decode()})")


def _pol(policy) -> int:
    """'fifo' | 'best_fit' | 'recent_fit' | 'random_fit', optionally with a
    '+literal' suffix, or the integer convgpu_policy_t [| LITERAL]."""
    if isinstance(policy, str):
        base, _, mode = policy.partition("+")
        if mode not in ("", "literal"):
            raise ConvgpuError(f"unknown dispatch reading {mode!r}")
        return POLICY[base] | (LITERAL if mode else 0)
    return int(policy)


def _ptr(t) -> Optional[int]:
    return None if t is None else t.data_ptr()


def _stream_handle(stream) -> int:
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return s.cuda_stream


# ---------------------------------------------------------------- data types
@dataclass
class Traces:
    """A batch of traces resident in device memory (C-ABI layout)."""
    arrival: "torch.Tensor"   # int32 view of uint32 [N, n]
    limit: "torch.Tensor"     # [N, n]
    op_delta: "torch.Tensor"  # [N, K, n]
    op_arg: "torch.Tensor"    # [N, K, n]
    trace_id_base: int = 0

    @property
    def count(self) -> int:
        return self.arrival.shape[0]

    @property
    def n(self) -> int:
        return self.arrival.shape[1]

    @property
    def K(self) -> int:
        return self.op_delta.shape[1]

    def nbytes(self) -> int:
        return sum(t.numel() * 4 for t in (self.arrival, self.limit, self.op_delta, self.op_arg))

    def struct(self, rand_seed=0, ovh=0, kernel="auto") -> TracesT:
        for t in (self.arrival, self.limit, self.op_delta, self.op_arg):
            if not t.is_contiguous():
                raise ConvgpuError("trace arrays must be contiguous")
        return TracesT(self.arrival.data_ptr(), self.limit.data_ptr(), self.op_delta.data_ptr(),
                       self.op_arg.data_ptr(), self.n, self.K, self.trace_id_base, rand_seed,
                       ovh, KERNEL[kernel])


def empty_traces(count: int, n: int, K: int, device="cuda", trace_id_base=0) -> Traces:
    import torch
    z = lambda *s: torch.empty(*s, dtype=torch.int32, device=device)  # noqa: E731
    return Traces(z(count, n), z(count, n), z(count, K, n), z(count, K, n), trace_id_base)


def traces_from_numpy(arrival, limit, delta, arg, device="cuda", trace_id_base=0) -> Traces:
    """Copy host numpy uint32 arrays ([N,n], [N,n], [N,K,n], [N,K,n]) to the device."""
    import torch
    f = lambda a: torch.from_numpy(np.ascontiguousarray(a, np.uint32).view(np.int32)).to(device)  # noqa: E731
    return Traces(f(arrival), f(limit), f(delta), f(arg), trace_id_base)


def gen_params_struct(g) -> GenParamsT:
    """From any object with the workload generator fields (workloads.GenParams)."""
    cm = list(g.class_mib)
    return GenParamsT(g.gen_seed, g.n, g.K, len(cm), (C.c_uint32 * 8)(*(cm + [0] * (8 - len(cm)))),
                      g.num, g.den, g.iat, g.dur_base, g.dur_step, g.dur_class_offset, g.dur_jit,
                      g.ovh)


def generate(g, trace_id_base: int, count: int, device="cuda", out: Optional[Traces] = None,
             stream=None) -> Traces:
    """Generate traces [trace_id_base, +count) on the device (convgpu_generate)."""
    t = out if out is not None else empty_traces(count, g.n, g.K, device, trace_id_base)
    t.trace_id_base = trace_id_base
    buf = BuffersT(t.arrival.data_ptr(), t.limit.data_ptr(), t.op_delta.data_ptr(),
                   t.op_arg.data_ptr())
    _check(lib().convgpu_generate(C.byref(gen_params_struct(g)), trace_id_base, count,
                                  C.byref(buf), _stream_handle(stream)), "convgpu_generate")
    return t


def wrap_ops(api, n: int, K: int, pitch_align: int = B200_PITCH_ALIGN, out=None, stream=None):
    """NEXT-3: map API-level records to scheduler op words on the device
    (convgpu_wrap_ops).  api: int32 tensor [N, K, n, 4] (convgpu_api_op_t
    records) on the GPU; returns (or fills) the int32 op_arg tensor [N, K, n]."""
    import torch
    if api.dim() != 4 or api.shape[1] != K or api.shape[2] != n or api.shape[3] != 4:
        raise ConvgpuError("api must be [N, K, n, 4] int32")
    N = api.shape[0]
    if out is None:
        out = torch.empty((N, K, n), dtype=torch.int32, device=api.device)
    _check(lib().convgpu_wrap_ops(api.data_ptr(), N, n, K, pitch_align, out.data_ptr(),
                                  _stream_handle(stream)), "convgpu_wrap_ops")
    return out


@dataclass
class ReplayOut:
    summary: Optional["torch.Tensor"] = None      # int64 [N, 5] (40-B records)
    stats: Optional["torch.Tensor"] = None        # int64 [12] (96 B)
    admit_tick: Optional["torch.Tensor"] = None   # int32 [N, n]
    admit_rank: Optional["torch.Tensor"] = None   # uint8 [N, n]
    wait: Optional["torch.Tensor"] = None
    finish: Optional["torch.Tensor"] = None
    range_digest: Optional["torch.Tensor"] = None  # int64 [R]
    range_size: int = 0
    admit_scratch: Optional["torch.Tensor"] = None  # int32 [N, n]: lets summary-only
    #                                                  launches use the compact kernel

    # host views (after synchronisation)
    def summary_np(self) -> np.ndarray:
        return self.summary.cpu().numpy().view(SUMMARY_DTYPE).reshape(-1)

    def stats_np(self) -> np.ndarray:
        return self.stats.cpu().numpy().view(STATS_DTYPE)[0]

    def full_np(self) -> dict:
        d = {}
        for f in ("admit_tick", "wait", "finish"):
            t = getattr(self, f)
            if t is not None:
                d[f] = t.cpu().numpy().view(np.uint32)
        if self.admit_rank is not None:
            d["admit_rank"] = self.admit_rank.cpu().numpy()
        return d


def alloc_out(count: int, n: int, device="cuda", full=True, summary=True, stats=True,
              range_count: int = 0, range_size: int = 0, scratch: bool = None) -> ReplayOut:
    """Device output buffers.  scratch (default: when per-container outputs are
    not requested) adds the admission scratch of convgpu_out_t, so that
    summary- / digest-only replays run on the compact lane kernel."""
    import torch
    o = ReplayOut()
    if scratch is None:
        scratch = not full
    if scratch and not full:
        o.admit_scratch = torch.empty(count, n, dtype=torch.int32, device=device)
    if summary:
        o.summary = torch.empty(count, 5, dtype=torch.int64, device=device)
    if stats:
        o.stats = torch.zeros(12, dtype=torch.int64, device=device)
    if full:
        o.admit_tick = torch.empty(count, n, dtype=torch.int32, device=device)
        o.admit_rank = torch.empty(count, n, dtype=torch.uint8, device=device)
        o.wait = torch.empty(count, n, dtype=torch.int32, device=device)
        o.finish = torch.empty(count, n, dtype=torch.int32, device=device)
    if range_count:
        o.range_digest = torch.zeros(range_count, dtype=torch.int64, device=device)
        o.range_size = range_size
    return o


def replay(traces: Traces, capacity: int, policy, out: ReplayOut, rand_seed: int = 0,
           ovh: int = 0, stream=None, kernel: str = "auto") -> ReplayOut:
    """Replay every trace of `traces` under `policy` (convgpu_replay).  Outputs
    go to the tensors of `out`; out.stats is accumulated (zero it first).
    kernel: "auto" | "warp" (warp per trace) | "lane" (lane per trace) |
    "lane16" (lane per trace, compact state; n = 64, K = 4, admit_tick or
    admit_scratch needed) | "lane16w" (the same, 17-bit layout first: for
    limits above 0xFFFE MiB)."""
    tr = traces.struct(rand_seed, ovh, kernel)
    o = OutT(_ptr(out.admit_tick), _ptr(out.admit_rank), _ptr(out.wait), _ptr(out.finish),
             _ptr(out.summary), _ptr(out.stats), _ptr(out.range_digest), out.range_size,
             _stream_handle(stream), _ptr(out.admit_scratch))
    _check(lib().convgpu_replay(C.byref(tr), traces.count, capacity, _pol(policy), C.byref(o)),
           "convgpu_replay")
    return out


def replay_host(arrival, limit, delta, arg, capacity: int, policies=("fifo",), *,
                trace_id_base=0, rand_seed=0, ovh=0, chunk: int = 1 << 15,
                summary: Optional[np.ndarray] = None, workspace=None, stream=None,
                kernel: str = "auto"):
    """End-to-end replay from HOST arrays (numpy or pinned torch; uint32/int32
    in the layouts of include/convgpu.h) through convgpu_replay_host: chunks
    are copied in, replayed under every policy in `policies` while resident,
    and summaries / statistics copied back.  Returns the statistics records
    (numpy STATS_DTYPE [n_policies], increasing policy id); fills
    `summary` ([n_policies, N] SUMMARY_DTYPE) if given."""
    import torch
    arrs = []
    for a in (arrival, limit, delta, arg):
        if isinstance(a, torch.Tensor):
            if a.is_cuda or not a.is_contiguous():
                raise ConvgpuError("replay_host expects contiguous host tensors")
            arrs.append(a)
        else:
            arrs.append(np.ascontiguousarray(a))
    ptr = lambda a: a.data_ptr() if isinstance(a, torch.Tensor) else a.ctypes.data  # noqa: E731
    N, n = arrs[0].shape[0], arrs[0].shape[1]
    K = arrs[2].shape[1]
    if isinstance(policies, (str, int)):
        policies = (policies,)
    mask = 0
    for q in policies:
        mask |= 1 << _pol(q)
    npol = bin(mask).count("1")
    tr = TracesT(ptr(arrs[0]), ptr(arrs[1]), ptr(arrs[2]), ptr(arrs[3]), n, K, trace_id_base,
                 rand_seed, ovh, KERNEL[kernel])
    need = host_workspace_bytes(n, K, chunk, npol)
    if workspace is None or workspace.numel() < need:
        workspace = torch.empty(need, dtype=torch.uint8, device="cuda")
    stats = np.zeros(npol, STATS_DTYPE)
    sp = None
    if summary is not None:
        assert summary.dtype == SUMMARY_DTYPE and summary.shape == (npol, N)
        assert summary.flags["C_CONTIGUOUS"]
        sp = summary.ctypes.data
    _check(lib().convgpu_replay_host(C.byref(tr), N, capacity, mask, sp, stats.ctypes.data,
                                     workspace.data_ptr(), workspace.numel(), chunk,
                                     _stream_handle(stream)), "convgpu_replay_host")
    return stats


def host_workspace_bytes(n: int, K: int, chunk: int, n_policies: int = 1, packed: bool = False) -> int:
    f = lib().convgpu_replay_host16_workspace if packed else lib().convgpu_replay_host_workspace
    return int(f(n, K, chunk, n_policies))


# ---------------------------------------------------------------- 16-bit format
@dataclass
class Traces16:
    """Traces in the compact 16-bit format of include/convgpu.h
    (convgpu_traces16_t): int16 views of u16 arrival / limit [N, n], op_size /
    op_delta [N, K, n]; uint8 op_kinds [N, n].  Device or (pinned) host."""
    arrival: "torch.Tensor"
    limit: "torch.Tensor"
    op_size: "torch.Tensor"
    op_delta: "torch.Tensor"
    op_kinds: "torch.Tensor"

    @property
    def count(self) -> int:
        return self.arrival.shape[0]

    @property
    def n(self) -> int:
        return self.arrival.shape[1]

    @property
    def K(self) -> int:
        return self.op_size.shape[1]

    def nbytes(self) -> int:
        return sum(t.numel() * t.element_size() for t in
                   (self.arrival, self.limit, self.op_size, self.op_delta, self.op_kinds))

    def pin(self) -> "Traces16":
        """A pinned host copy (the e2e input)."""
        import torch
        cp = lambda t: torch.empty(t.shape, dtype=t.dtype, pin_memory=True).copy_(t)  # noqa: E731
        return Traces16(*(cp(t) for t in (self.arrival, self.limit, self.op_size, self.op_delta,
                                          self.op_kinds)))


def pack16(traces: Traces, stream=None) -> tuple:
    """Pack device traces into the 16-bit format on the device
    (convgpu_pack16).  Returns (Traces16, out_of_range tensor): the packed
    batch is exact iff out_of_range (int64[1], read after synchronising) is 0."""
    import torch
    N, n, K = traces.count, traces.n, traces.K
    dev = traces.arrival.device
    e = lambda *sh: torch.empty(*sh, dtype=torch.int16, device=dev)  # noqa: E731
    t16 = Traces16(e(N, n), e(N, n), e(N, K, n), e(N, K, n),
                   torch.empty(N, n, dtype=torch.uint8, device=dev))
    oor = torch.zeros(1, dtype=torch.int64, device=dev)
    buf = Buffers16T(t16.arrival.data_ptr(), t16.limit.data_ptr(), t16.op_size.data_ptr(),
                     t16.op_delta.data_ptr(), t16.op_kinds.data_ptr())
    _check(lib().convgpu_pack16(C.byref(traces.struct()), N, C.byref(buf), oor.data_ptr(),
                                _stream_handle(stream)), "convgpu_pack16")
    return t16, oor


def replay_host16(t16: Traces16, capacity: int, policies=("fifo",), *, trace_id_base=0,
                  rand_seed=0, ovh=0, chunk: int = 1 << 15, summary: Optional[np.ndarray] = None,
                  workspace=None, stream=None, kernel: str = "auto"):
    """End-to-end replay of HOST traces in the 16-bit format
    (convgpu_replay_host16); as replay_host otherwise."""
    import torch
    for t in (t16.arrival, t16.limit, t16.op_size, t16.op_delta, t16.op_kinds):
        if t.is_cuda or not t.is_contiguous():
            raise ConvgpuError("replay_host16 expects contiguous host tensors")
    if isinstance(policies, (str, int)):
        policies = (policies,)
    mask = 0
    for q in policies:
        mask |= 1 << _pol(q)
    npol = bin(mask).count("1")
    N, n, K = t16.count, t16.n, t16.K
    tr = Traces16T(t16.arrival.data_ptr(), t16.limit.data_ptr(), t16.op_size.data_ptr(),
                   t16.op_delta.data_ptr(), t16.op_kinds.data_ptr(), n, K, trace_id_base,
                   rand_seed, ovh, KERNEL[kernel])
    need = host_workspace_bytes(n, K, chunk, npol, packed=True)
    if workspace is None or workspace.numel() < need:
        workspace = torch.empty(need, dtype=torch.uint8, device="cuda")
    stats = np.zeros(npol, STATS_DTYPE)
    sp = None
    if summary is not None:
        assert summary.dtype == SUMMARY_DTYPE and summary.shape == (npol, N)
        assert summary.flags["C_CONTIGUOUS"]
        sp = summary.ctypes.data
    _check(lib().convgpu_replay_host16(C.byref(tr), N, capacity, mask, sp, stats.ctypes.data,
                                       workspace.data_ptr(), workspace.numel(), chunk,
                                       _stream_handle(stream)), "convgpu_replay_host16")
    return stats


def stats_dict(rec) -> dict:
    d = {k: int(rec[k]) for k in STATS_DTYPE.names if k != "flag_count"}
    d["flag_count"] = [int(x) for x in rec["flag_count"]]
    return d
