#!/usr/bin/env python
"""Probe the CUDA runtime's pitched-allocation sizes on this GPU (NEXT-3, the
wrapper-side size semantics of P:106-108).  Prints the device properties the
wrapper module would read on its first cudaMallocPitch and the pitch
cudaMallocPitch / cudaMalloc3D return for a sweep of row widths, as JSON.

  python scripts/probe_pitch.py > gpurun_out/pitch_probe.json
"""
import json
import sys


def main():
    from cuda.bindings import runtime as rt
    err, prop = rt.cudaGetDeviceProperties(0)
    assert err == rt.cudaError_t.cudaSuccess, err
    out = {"device": prop.name.decode() if isinstance(prop.name, bytes) else str(prop.name),
           "texturePitchAlignment": int(prop.texturePitchAlignment),
           "textureAlignment": int(prop.textureAlignment),
           "memPitch": int(prop.memPitch), "pitch": [], "pitch3d": []}
    widths = list(range(1, 2049)) + [2 ** e + d for e in range(11, 21) for d in (-1, 0, 1)]
    for w in widths:
        err, ptr, pitch = rt.cudaMallocPitch(w, 3)
        assert err == rt.cudaError_t.cudaSuccess, (w, err)
        out["pitch"].append([w, int(pitch)])
        rt.cudaFree(ptr)
    for w in (1, 100, 511, 512, 513, 1000, 4096, 5000):
        for h, d in ((1, 1), (7, 3)):
            err, pp = rt.cudaMalloc3D(rt.make_cudaExtent(w, h, d))
            assert err == rt.cudaError_t.cudaSuccess, (w, err)
            out["pitch3d"].append([w, h, d, int(pp.pitch)])
            rt.cudaFree(pp.ptr)
    json.dump(out, sys.stdout)
    print()


if __name__ == "__main__":
    main()
