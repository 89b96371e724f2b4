"""NEXT-4: the live control plane's Python side (include/convgpu_ctl.h).

`Daemon` starts and stops `convgpud` (the native scheduler daemon built by
build.py); `Client` is one process of one container speaking the 32-byte
message protocol.  The wrapper module itself is native
(`libconvgpu_shim.so`, LD_PRELOAD); this module is for operators, drivers and
tests.
"""
from __future__ import annotations

import os
import socket
import struct
import subprocess
import time

HERE = os.path.dirname(os.path.abspath(__file__))
DAEMON = os.path.join(HERE, "convgpud")
SHIM = os.path.join(HERE, "libconvgpu_shim.so")

HELLO, ALLOC, ALLOC_DONE, ALLOC_FAIL, FREE, FREE_BYTES, MEMINFO, EXIT, INFO, STATS, SYNC = range(1, 12)
OK, REJECT, INVALID, PROTOCOL = range(4)
NONE64 = (1 << 64) - 1
_MSG = struct.Struct("=IIQQQ")
_REP = struct.Struct("=iIQQQ")
POLICIES = ("fifo", "best_fit", "recent_fit", "random_fit")


class Daemon:
    """A convgpud process on a UNIX socket path (units as given)."""

    def __init__(self, path: str, capacity: int, policy: str = "fifo", overhead: int = 0,
                 seed: int = 0, tid: int = 0):
        if not os.path.exists(DAEMON):
            raise RuntimeError(f"{DAEMON} missing: run __graft_entry__.build()")
        self.path = path
        self.proc = subprocess.Popen(
            [DAEMON, "--socket", path, "--capacity", str(capacity), "--policy", policy,
             "--overhead", str(overhead), "--seed", str(seed), "--tid", str(tid)],
            stdout=subprocess.PIPE, stderr=subprocess.PIPE, text=True)
        line = self.proc.stdout.readline()
        if not line.startswith("convgpud ready"):
            raise RuntimeError(f"convgpud failed: {line!r} {self.proc.stderr.read()}")

    def close(self):
        if self.proc.poll() is None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
        try:
            os.unlink(self.path)
        except OSError:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()


class Client:
    """One connection (= one process of one container, or a control link)."""

    def __init__(self, path: str, pid: int | None = None):
        self.s = socket.socket(socket.AF_UNIX, socket.SOCK_STREAM)
        for _ in range(200):
            try:
                self.s.connect(path)
                break
            except (FileNotFoundError, ConnectionRefusedError):
                time.sleep(0.01)
        else:
            raise RuntimeError(f"cannot connect to {path}")
        self.pid = os.getpid() if pid is None else pid

    def send(self, typ: int, a: int = 0, b: int = 0, c: int = 0):
        self.s.sendall(_MSG.pack(typ, self.pid & 0xFFFFFFFF, a, b, c))

    def recv(self, block: bool = True):
        """One reply (status, type, a, b, c), or None if none is pending and
        block is False."""
        self.s.setblocking(block)
        try:
            buf = b""
            while len(buf) < _REP.size:
                chunk = self.s.recv(_REP.size - len(buf))
                if not chunk:
                    raise ConnectionError("convgpud closed the connection")
                buf += chunk
                self.s.setblocking(True)
            return _REP.unpack(buf)
        except BlockingIOError:
            return None
        finally:
            self.s.setblocking(True)

    def call(self, typ: int, a: int = 0, b: int = 0, c: int = 0):
        self.send(typ, a, b, c)
        return self.recv()

    def close(self):
        self.s.close()
