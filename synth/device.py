"""Device-side generation of the config-5 batch (8,192 meshes, ~176 M nodes,
~2.5 G nnz) -- too large for numpy in a benchmark setup.  Bit-identical to
synth.c5_matrix(k, N) (tests/test_gpu_parity.py::test_c5_device_generator).
Input generation only: no arithmetic of the RCM method."""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from . import c5_dims, c5_sizes

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "csrc", "synth_gen.cu")
_LIB = os.path.join(_HERE, "libsynth_gen.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                               "-std=c++17", "-Xcompiler", "-fPIC", "-cudart", "static", "-shared",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        vp = ctypes.c_void_p
        lib.synth_c5_degrees.argtypes = [vp, vp, ctypes.c_int, ctypes.c_longlong, vp, vp]
        lib.synth_c5_fill.argtypes = [vp, vp, vp, ctypes.c_int, ctypes.c_longlong, vp, vp, vp]
        _lib = lib
    return _lib


def c5_specs(mats, sizes):
    """(kind, nx, ny, nz, gid) per selected matrix, plus n_k and nnz_k."""
    spec = np.zeros((len(mats), 5), np.int32)
    n = np.zeros(len(mats), np.int64)
    nnz = np.zeros(len(mats), np.int64)
    for i, k in enumerate(mats):
        d = c5_dims(int(k), int(sizes[k]))
        if len(d) == 2:
            w, h = d
            spec[i] = (2, w, h, 1, k)
            n[i] = w * h
            nnz[i] = w * h + 2 * ((w - 1) * h + w * (h - 1))
        else:
            a, b, c = d
            spec[i] = (3, a, b, c, k)
            n[i] = a * b * c
            nnz[i] = (3 * a - 2) * (3 * b - 2) * (3 * c - 2)
    return spec, n, nnz


def c5_generate(mats=None, num: int = 8192, seed: int = 5, lo: float = 1e3, hi: float = 1e5,
                device="cuda"):
    """Generate the selected matrices (default: all) of the config-5 batch on the
    device.  Returns a dict of torch tensors in rcm_reorder_batched layout."""
    import torch
    sizes = c5_sizes(num, seed, lo, hi)
    mats = np.arange(num) if mats is None else np.asarray(mats, dtype=np.int64)
    spec, n, nnz = c5_specs(mats, sizes)
    node_off = np.zeros(len(mats) + 1, np.int64)
    nnz_off = np.zeros(len(mats) + 1, np.int64)
    node_off[1:] = np.cumsum(n)
    nnz_off[1:] = np.cumsum(nnz)
    total, total_nnz, m = int(node_off[-1]), int(nnz_off[-1]), len(mats)
    dev = torch.device(device)
    stream = torch.cuda.current_stream(dev).cuda_stream
    specs_d = torch.from_numpy(spec).to(dev)
    node_off_d = torch.from_numpy(node_off).to(dev)
    nnz_off_d = torch.from_numpy(nnz_off).to(dev)
    deg = torch.empty(total, dtype=torch.int32, device=dev)
    lib = _load()
    # the kernels take the global matrix id from spec[:, 4] through the MatSpec layout
    rc = lib.synth_c5_degrees(specs_d.data_ptr(), node_off_d.data_ptr(), m, total, deg.data_ptr(), stream)
    assert rc == 0, rc
    cs = torch.zeros(total + 1, dtype=torch.int64, device=dev)
    torch.cumsum(deg.to(torch.int64), 0, out=cs[1:])
    assert int(cs[-1].item()) == total_nnz
    counts = torch.from_numpy(n + 1).to(dev)
    kk = torch.repeat_interleave(torch.arange(m, device=dev), counts)
    pos = torch.arange(total + m, device=dev, dtype=torch.int64) - (node_off_d[kk] + kk)
    rp = (cs[node_off_d[kk] + pos] - cs[node_off_d[kk]]).to(torch.int32)
    col = torch.empty(total_nnz, dtype=torch.int32, device=dev)
    rc = lib.synth_c5_fill(specs_d.data_ptr(), node_off_d.data_ptr(), nnz_off_d.data_ptr(), m, total,
                           rp.data_ptr(), col.data_ptr(), stream)
    assert rc == 0, rc
    del deg, cs, kk, pos
    return {"mats": mats, "sizes": sizes[mats], "node_off": node_off_d, "nnz_off": nnz_off_d,
            "node_off_h": node_off, "nnz_off_h": nnz_off, "row_ptr_local": rp, "col_idx_local": col,
            "total": total, "total_nnz": total_nnz}
