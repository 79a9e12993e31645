"""GPU twin of inputs/graphs.py (input generation only; see tqgen.cu).

Builds the same CSR as `inputs.graphs` bit for bit, directly in device memory,
for the large configs (Kronecker scale 24/26, grid 4096^2) where numpy is too
slow. Returns torch CUDA tensors (row_ptr int64[V+1], col int32[nnz]).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "csrc", "tqgen.cu")
LIB = os.path.join(HERE, "libtqgen.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call([NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-std=c++17",
                               "-Xcompiler", "-fPIC", "-shared", "-o", tmp, SRC])
        os.replace(tmp, LIB)
    return LIB


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB):
            raise ImportError(f"{LIB} missing; run inputs.gpu.build()")
        L = ctypes.CDLL(LIB)
        vp, i64 = ctypes.c_void_p, ctypes.c_int64
        L.tqgen_kron_keys.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_uint64, vp, vp]
        L.tqgen_grid_keys.argtypes = [i64, i64, vp, vp]
        L.tqgen_tree4_keys.argtypes = [i64, vp, vp]
        L.tqgen_sort_unique.argtypes = [vp, vp, i64, ctypes.POINTER(i64), vp]
        L.tqgen_keys_to_csr.argtypes = [vp, i64, i64, vp, vp, vp]
        L.tqgen_edge_weights.argtypes = [vp, vp, i64, ctypes.c_uint64, ctypes.c_uint32, vp, vp]
        for f in ("tqgen_kron_keys", "tqgen_grid_keys", "tqgen_tree4_keys", "tqgen_sort_unique",
                  "tqgen_keys_to_csr", "tqgen_edge_weights"):
            getattr(L, f).restype = ctypes.c_int
        _lib = L
    return _lib


def _finish(keys, nv: int, device):
    import torch
    alt = torch.empty_like(keys)
    n = ctypes.c_int64()
    s = torch.cuda.current_stream(device).cuda_stream
    if lib().tqgen_sort_unique(keys.data_ptr(), alt.data_ptr(), keys.numel(), ctypes.byref(n), s):
        raise RuntimeError("tqgen_sort_unique failed")
    del alt
    nnz = n.value
    row_ptr = torch.empty(nv + 1, dtype=torch.int64, device=device)
    col = torch.empty(max(nnz, 1), dtype=torch.int32, device=device)
    if lib().tqgen_keys_to_csr(keys.data_ptr(), nnz, nv, row_ptr.data_ptr(), col.data_ptr(), s):
        raise RuntimeError("tqgen_keys_to_csr failed")
    torch.cuda.synchronize(device)
    return row_ptr, col[:nnz]


def kronecker_csr_cuda(scale: int, edgefactor: int = 16, seed: int = 1, device="cuda:0"):
    import torch
    m = edgefactor << scale
    keys = torch.empty(2 * m, dtype=torch.int64, device=device)
    s = torch.cuda.current_stream(device).cuda_stream
    if lib().tqgen_kron_keys(scale, edgefactor, seed & 0xFFFFFFFFFFFFFFFF, keys.data_ptr(), s):
        raise RuntimeError("tqgen_kron_keys failed")
    return _finish(keys, 1 << scale, device)


def grid_csr_cuda(rows: int, cols: int | None = None, device="cuda:0"):
    import torch
    cols = rows if cols is None else cols
    keys = torch.empty(4 * rows * cols, dtype=torch.int64, device=device)
    s = torch.cuda.current_stream(device).cuda_stream
    if lib().tqgen_grid_keys(rows, cols, keys.data_ptr(), s):
        raise RuntimeError("tqgen_grid_keys failed")
    return _finish(keys, rows * cols, device)


def edge_weights_cuda(row_ptr, col, seed: int, wmax: int = 255):
    """Twin of inputs.graphs.edge_weights on device tensors."""
    import torch
    w = torch.empty(col.numel(), dtype=torch.int32, device=col.device)
    s = torch.cuda.current_stream(col.device).cuda_stream
    if lib().tqgen_edge_weights(row_ptr.data_ptr(), col.data_ptr(), row_ptr.numel() - 1,
                                seed & 0xFFFFFFFFFFFFFFFF, wmax, w.data_ptr(), s):
        raise RuntimeError("tqgen_edge_weights failed")
    return w


def tree4_csr_cuda(n: int, device="cuda:0"):
    import torch
    keys = torch.empty(2 * n, dtype=torch.int64, device=device)
    s = torch.cuda.current_stream(device).cuda_stream
    if lib().tqgen_tree4_keys(n, keys.data_ptr(), s):
        raise RuntimeError("tqgen_tree4_keys failed")
    return _finish(keys, n, device)
