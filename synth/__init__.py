"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This module holds only input generation (no SpMV, permutation or reordering
arithmetic).  ``synth/csrc/synth.cpp`` is the fast generator (OpenMP);
``synth/gen.py`` is the same definition as plain loops for tiny sizes.

Workload recipe:

======  ===============================================================
C1      RMAT scale 16, edge factor 16, (a,b,c,d)=(.57,.19,.19,.05), unscrambled
C2      SBM 4096 communities x 1024, 16 distinct columns/row, p_in .97, scrambled
C3      RMAT scale 26, edge factor 16, unscrambled
C4      27-point stencil 464^3, Dirichlet, random relabel
C5      Graph500 Kronecker scale 28, ef 16, vertex scramble, values U(0,1]
======  ===============================================================
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import weakref
from dataclasses import dataclass

import numpy as np

from . import gen  # noqa: F401  (reference loops)

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libsynth.so")
_SRC = os.path.join(_HERE, "csrc", "synth.cpp")
_SO_GPU = os.path.join(_HERE, "libsynth_gpu.so")
_SRC_GPU = os.path.join(_HERE, "csrc", "synth_gpu.cu")

BASE_SEED = 20230423


def build(force: bool = False) -> str:
    """Compile libsynth.so (host C++, OpenMP) and libsynth_gpu.so (the RMAT /
    Kronecker generator on the GPU, sm_100a) in-tree."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        cmd = ["g++", "-O3", "-march=x86-64-v2", "-std=c++17", "-fopenmp", "-shared",
               "-fPIC", "-o", _SO, _SRC]
        subprocess.check_call(cmd)
    if force or not os.path.exists(_SO_GPU) or \
            os.path.getmtime(_SO_GPU) < os.path.getmtime(_SRC_GPU):
        nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
        cmd = [nvcc, "-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a",
               "-lineinfo", "-Xcompiler", "-fPIC", "-shared", "-o", _SO_GPU + ".tmp", _SRC_GPU,
               "-lcudart"]
        subprocess.check_call(cmd)
        os.replace(_SO_GPU + ".tmp", _SO_GPU)
    return _SO


class _Csr(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("row_ptr", ctypes.c_void_p), ("col", ctypes.c_void_p),
                ("val", ctypes.c_void_p)]


_lib = None
_libc = ctypes.CDLL(None)
_libc.free.argtypes = [ctypes.c_void_p]


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        u64, i64, i32, dbl = ctypes.c_uint64, ctypes.c_int64, ctypes.c_int, ctypes.c_double
        P = ctypes.POINTER(_Csr)
        L.synth_rmat.argtypes = [i32, i64, u64, dbl, dbl, dbl, i32, u64, i32, u64, P]
        L.synth_sbm.argtypes = [i64, i64, i32, dbl, u64, i32, u64, i32, u64, P]
        L.synth_stencil27.argtypes = [i64, i32, i32, u64, i32, u64, P]
        L.synth_vector.argtypes = [i64, u64, i32, ctypes.c_void_p]
        L.synth_scramble.argtypes = [i64, u64, ctypes.c_void_p]
        L.synth_h1.argtypes = [u64, u64]
        L.synth_h1.restype = u64
        L.synth_h2.argtypes = [u64, u64, u64]
        L.synth_h2.restype = u64
        L.synth_threads.restype = i32
        _lib = L
    return _lib


def _own(addr: int, n: int, ctype, dtype) -> np.ndarray:
    """Wrap malloc'd memory as a numpy array that frees it when collected."""
    n = max(int(n), 0)
    if n == 0:
        _libc.free(addr)
        return np.zeros(0, dtype)
    buf = (ctype * n).from_address(addr)
    weakref.finalize(buf, _libc.free, ctypes.c_void_p(addr))
    return np.frombuffer(buf, dtype=dtype)


@dataclass
class Csr:
    """Host CSR: row_ptr int64[n+1], col int32[nnz], val float32[nnz]."""
    n: int
    row_ptr: np.ndarray
    col: np.ndarray
    val: np.ndarray

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])


def _take(m: _Csr) -> Csr:
    return Csr(int(m.n), _own(m.row_ptr, m.n + 1, ctypes.c_int64, np.int64),
               _own(m.col, m.nnz, ctypes.c_int32, np.int32),
               _own(m.val, m.nnz, ctypes.c_float, np.float32))


VAL_SYM, VAL_POS, VAL_ONES = 0, 1, 2


def rmat(scale, edge_factor=16, seed=1, a=0.57, b=0.19, c=0.19, scramble=False,
         seed_scr=0, valmode=VAL_SYM, seed_v=0) -> Csr:
    m = _Csr()
    rc = lib().synth_rmat(scale, edge_factor, seed, a, b, c, int(scramble), seed_scr,
                          valmode, seed_v, ctypes.byref(m))
    if rc:
        raise RuntimeError(f"synth_rmat failed ({rc})")
    return _take(m)


def sbm(n_comm, comm_size, deg=16, p_in=0.97, seed=1, scramble=True, seed_scr=0,
        valmode=VAL_SYM, seed_v=0) -> Csr:
    m = _Csr()
    rc = lib().synth_sbm(n_comm, comm_size, deg, p_in, seed, int(scramble), seed_scr,
                         valmode, seed_v, ctypes.byref(m))
    if rc:
        raise RuntimeError(f"synth_sbm failed ({rc})")
    return _take(m)


def stencil27(nx, periodic=False, relabel=True, seed_scr=0, valmode=VAL_SYM,
              seed_v=0) -> Csr:
    m = _Csr()
    rc = lib().synth_stencil27(nx, int(periodic), int(relabel), seed_scr, valmode,
                               seed_v, ctypes.byref(m))
    if rc:
        raise RuntimeError(f"synth_stencil27 failed ({rc})")
    return _take(m)


class _GpuCsr(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("row_ptr", ctypes.c_void_p), ("col", ctypes.c_void_p),
                ("val", ctypes.c_void_p)]


_lib_gpu = None


def lib_gpu():
    global _lib_gpu
    if _lib_gpu is None:
        build()
        L = ctypes.CDLL(_SO_GPU)
        u64, i64, i32, dbl = ctypes.c_uint64, ctypes.c_int64, ctypes.c_int, ctypes.c_double
        L.synth_rmat_gpu.argtypes = [i32, i64, u64, dbl, dbl, dbl, i32, u64, i32, u64, i32,
                                     ctypes.POINTER(_GpuCsr)]
        L.synth_gpu_free.argtypes = [ctypes.POINTER(_GpuCsr)]
        L.synth_gpu_error.restype = ctypes.c_char_p
        _lib_gpu = L
    return _lib_gpu


class _DevArray:
    """Owner of one cudaMalloc'ed array of a _GpuCsr (freed with the last view)."""

    def __init__(self, owner, ptr, n, typestr):
        self._owner = owner
        self.__cuda_array_interface__ = {"shape": (int(n),), "typestr": typestr,
                                         "data": (int(ptr) if ptr else 0, False), "version": 3}


class _GpuOwner:
    def __init__(self, m):
        self.m = m

    def __del__(self):
        try:
            lib_gpu().synth_gpu_free(ctypes.byref(self.m))
        except Exception:
            pass


@dataclass
class DeviceCsr:
    """CSR on a CUDA device (torch tensors): row_ptr int64[n+1], col int32[nnz],
    val float32[nnz]."""
    n: int
    row_ptr: object
    col: object
    val: object

    @property
    def nnz(self) -> int:
        return int(self.col.numel())

    def to_host(self) -> Csr:
        return Csr(self.n, self.row_ptr.cpu().numpy(), self.col.cpu().numpy(),
                   self.val.cpu().numpy())


def rmat_gpu(scale, edge_factor=16, seed=1, a=0.57, b=0.19, c=0.19, scramble=False,
             seed_scr=0, valmode=VAL_SYM, seed_v=0, device=0) -> DeviceCsr:
    """rmat() generated on CUDA device `device` (bit-identical CSR)."""
    import torch
    m = _GpuCsr()
    rc = lib_gpu().synth_rmat_gpu(scale, edge_factor, seed, a, b, c, int(scramble), seed_scr,
                                  valmode, seed_v, int(device), ctypes.byref(m))
    if rc:
        raise RuntimeError(f"synth_rmat_gpu failed ({rc}): {lib_gpu().synth_gpu_error().decode()}")
    own = _GpuOwner(m)
    dev = torch.device("cuda", int(device))
    t = lambda p, k, ts: torch.as_tensor(_DevArray(own, p, k, ts), device=dev)  # noqa: E731
    nnz = int(m.nnz)
    return DeviceCsr(int(m.n), t(m.row_ptr, m.n + 1, "<i8"),
                     t(m.col, nnz, "<i4") if nnz else torch.zeros(0, dtype=torch.int32, device=dev),
                     t(m.val, nnz, "<f4") if nnz else torch.zeros(0, dtype=torch.float32, device=dev))


def vector(n, seed_x, mode=VAL_SYM) -> np.ndarray:
    out = np.empty(n, np.float32)
    lib().synth_vector(n, seed_x, mode, out.ctypes.data)
    return out


def scramble_table(n, seed_scr) -> np.ndarray:
    out = np.empty(n, np.int64)
    lib().synth_scramble(n, seed_scr, out.ctypes.data)
    return out


def seeds(k: int):
    """Sub-seeds of config k: (edges, values, x, scramble)."""
    s = BASE_SEED + k
    return tuple(gen.h1(s, i) for i in (1, 2, 3, 4))


@dataclass
class Workload:
    name: str
    A: Csr
    x: np.ndarray
    planted: np.ndarray | None = None   # ground-truth order (SBM communities, stencil
                                        # grid), perm[old] = new; reference only


def config_gpu(k: int, device=0, small: bool = False):
    """The RMAT / Kronecker workloads (k = 1, 3, 5) generated on the GPU:
    (name, DeviceCsr, x host float32) -- the same matrix as config(k)."""
    se, sv, sx, ss = seeds(k)
    if k == 1:
        sc = 12 if small else 16
        A = rmat_gpu(sc, 16, se, seed_v=sv, device=device)
        return f"rmat{sc}", A, vector(A.n, sx)
    if k == 3:
        sc = 16 if small else 26
        A = rmat_gpu(sc, 16, se, seed_v=sv, device=device)
        return f"rmat{sc}", A, vector(A.n, sx)
    if k == 5:
        sc = 14 if small else 28
        A = rmat_gpu(sc, 16, se, scramble=True, seed_scr=ss, valmode=VAL_POS, seed_v=sv,
                     device=device)
        return f"kron{sc}", A, np.full(A.n, np.float32(1.0 / np.sqrt(A.n)), np.float32)
    raise ValueError(f"config {k} has no GPU generator")


def config(k: int, small: bool = False) -> Workload:
    """The five SURVEY.md §8(d) workloads; ``small`` gives a same-shaped
    reduced instance for parity tests."""
    se, sv, sx, ss = seeds(k)
    if k == 1:
        sc = 12 if small else 16
        A = rmat(sc, 16, se, seed_v=sv)
        return Workload(f"rmat{sc}", A, vector(A.n, sx))
    if k == 2:
        nc = 16 if small else 4096
        A = sbm(nc, 1024, 16, 0.97, se, True, ss, VAL_SYM, sv)
        planted = np.empty(A.n, np.int64)
        planted[scramble_table(A.n, ss)] = np.arange(A.n)
        return Workload(f"sbm{nc}x1024", A, vector(A.n, sx), planted)
    if k == 3:
        sc = 16 if small else 26
        A = rmat(sc, 16, se, seed_v=sv)
        return Workload(f"rmat{sc}", A, vector(A.n, sx))
    if k == 4:
        nx = 24 if small else 464
        A = stencil27(nx, False, True, ss, VAL_SYM, sv)
        planted = np.empty(A.n, np.int64)   # lexicographic grid order
        planted[scramble_table(A.n, ss)] = np.arange(A.n)
        return Workload(f"stencil27_{nx}", A, vector(A.n, sx), planted)
    if k == 5:
        sc = 14 if small else 28
        A = rmat(sc, 16, se, scramble=True, seed_scr=ss, valmode=VAL_POS, seed_v=sv)
        x = np.full(A.n, np.float32(1.0 / np.sqrt(A.n)), np.float32)
        return Workload(f"kron{sc}", A, x)
    raise ValueError(k)
