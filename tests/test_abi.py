"""The C-ABI library builds, loads and exports every symbol include/convgpu.h
declares; argument validation that precedes any device work (CPU only)."""
import ctypes as C
import errno
import os
import re

import pytest

import paper_conf_cluster_kangjkkk17_b200 as cg
from paper_conf_cluster_kangjkkk17_b200 import build as B

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def so():
    B.build()
    return cg.lib()


def declared_functions():
    src = open(os.path.join(ROOT, "include", "convgpu.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(convgpu_\w+)\s*\(", src)))


def test_exports_every_declared_symbol(so):
    names = declared_functions()
    assert len(names) >= 7
    for name in names:
        assert hasattr(so, name), name
    assert set(names) == set(cg.EXPORTS)


def test_nm_lists_symbols_as_extern_c(so):
    import subprocess
    out = subprocess.run(["nm", "-D", "--defined-only", cg.SO_PATH], capture_output=True,
                         text=True).stdout
    for name in declared_functions():
        assert re.search(r"\sT\s%s$" % name, out, re.M), name


def test_version_and_strerror(so):
    assert so.convgpu_abi_version() == 5
    assert so.convgpu_launches_per_call() == 3
    assert b"invalid" in so.convgpu_strerror(-errno.EINVAL)
    assert b"sm_100" in so.convgpu_strerror(-errno.ENODEV)


def test_workspace_size(so):
    w = so.convgpu_replay_host_workspace(64, 4, 1000, 1)
    assert w >= 2 * 1000 * 64 * 4 * 10 + 2 * 1000 * 40 + 96
    assert so.convgpu_replay_host_workspace(64, 4, 1000, 4) >= w + 6 * 1000 * 40 + 3 * 96


def _traces(**kw):
    t = cg.TracesT(1, 1, 1, 1, 64, 4, 0, 0, 0, 0)
    for k, v in kw.items():
        setattr(t, k, v)
    return t


@pytest.mark.parametrize("kw", [dict(n_containers=0), dict(n_containers=65), dict(n_ops=0),
                                dict(n_ops=9), dict(arrival=None), dict(op_arg=None),
                                dict(kernel_variant=5), dict(ctx_overhead_mib=1 << 30),
                                dict(kernel_variant=3, n_containers=16)])
def test_replay_rejects_bad_shape_before_touching_the_device(so, kw):
    out = cg.OutT()
    assert so.convgpu_replay(C.byref(_traces(**kw)), 10, 1000, 0, C.byref(out)) == -errno.EINVAL


@pytest.mark.parametrize("cap,policy", [(0, 0), (1 << 26, 0), (100, -1), (100, 4)])
def test_replay_rejects_bad_capacity_policy(so, cap, policy):
    out = cg.OutT()
    assert so.convgpu_replay(C.byref(_traces()), 10, cap, policy, C.byref(out)) == -errno.EINVAL


def test_replay_null_struct(so):
    assert so.convgpu_replay(None, 1, 100, 0, None) == -errno.EINVAL
    assert so.convgpu_replay(C.byref(_traces()), 1, 100, 0, None) == -errno.EINVAL


def test_range_digest_requires_size(so):
    out = cg.OutT()
    out.range_digest = 8
    out.range_size = 0
    assert so.convgpu_replay(C.byref(_traces()), 1, 100, 0, C.byref(out)) == -errno.EINVAL


def test_generate_rejects_bad_params(so):
    p = cg.GenParamsT()
    p.n_containers, p.n_ops, p.n_classes, p.den = 64, 3, 6, 1
    buf = cg.BuffersT(1, 1, 1, 1)
    assert so.convgpu_generate(C.byref(p), 0, 10, C.byref(buf), None) == -errno.EINVAL
    p.n_ops, p.den = 4, 0
    assert so.convgpu_generate(C.byref(p), 0, 10, C.byref(buf), None) == -errno.EINVAL


def test_no_device_is_enodev_not_a_fallback(so):
    """Without a GPU the library refuses (no CPU fallback)."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    out = cg.OutT()
    rc = so.convgpu_replay(C.byref(_traces()), 1, 100, 0, C.byref(out))
    assert rc in (-errno.ENODEV, -errno.EIO)


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_cluster_kangjkkk17_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".c")):
                txt = open(os.path.join(dp, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
                assert "oracle.h" not in txt and "liboracle" not in txt, f


def test_missing_extension_fails_loudly(monkeypatch, tmp_path):
    """No CPU fallback: without libconvgpu.so every call raises."""
    monkeypatch.setattr(cg, "SO_PATH", str(tmp_path / "missing.so"))
    monkeypatch.setattr(cg, "_lib", None)
    with pytest.raises(cg.ConvgpuError):
        cg.lib()


def _traces16(**kw):
    t = cg.Traces16T(1, 1, 1, 1, 1, 64, 4, 0, 0, 0, 0)
    for k, v in kw.items():
        setattr(t, k, v)
    return t


@pytest.mark.parametrize("kw", [dict(n_ops=5), dict(n_ops=0), dict(n_containers=65),
                                dict(op_kinds=None), dict(arrival=None), dict(kernel_variant=5)])
def test_replay_host16_rejects_bad_shape_before_touching_the_device(so, kw):
    st = (C.c_uint8 * 96)()
    assert so.convgpu_replay_host16(C.byref(_traces16(**kw)), 10, 1000, 1, None, st, 1, 1 << 30,
                                    16, None) == -errno.EINVAL


def test_replay_host16_rejects_empty_mask_and_null(so):
    st = (C.c_uint8 * 96)()
    assert so.convgpu_replay_host16(C.byref(_traces16()), 10, 1000, 0, None, st, 1, 1 << 30,
                                    16, None) == -errno.EINVAL
    assert so.convgpu_replay_host16(None, 10, 1000, 1, None, st, 1, 1 << 30, 16,
                                    None) == -errno.EINVAL


def test_pack16_rejects_bad_shape(so):
    buf = cg.Buffers16T(1, 1, 1, 1, 1)
    assert so.convgpu_pack16(C.byref(_traces(n_ops=5)), 10, C.byref(buf), None, None) == -errno.EINVAL
    assert so.convgpu_pack16(C.byref(_traces(n_containers=0)), 10, C.byref(buf), None,
                             None) == -errno.EINVAL
    assert so.convgpu_pack16(None, 10, C.byref(buf), None, None) == -errno.EINVAL


def test_workspace16_size(so):
    """The 16-bit path holds two 16-bit copy-in sets and one 32-bit unpack
    target instead of two 32-bit sets."""
    w32 = so.convgpu_replay_host_workspace(64, 4, 1000, 4)
    w16 = so.convgpu_replay_host16_workspace(64, 4, 1000, 4)
    assert w16 >= w32 - 1000 * 64 * 40 + 2 * 1000 * 64 * 21
