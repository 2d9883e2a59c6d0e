"""Thin ctypes binding of include/spmv.h (argument marshalling only).

Every step of the path runs in libspmv.so; torch supplies device memory and
streams.  There is no fallback: if the library is missing or a call fails,
an exception is raised.
"""
from __future__ import annotations

import ctypes
import os
import re
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
SO_PATH = os.path.join(_HERE, "libspmv.so")
HEADER = os.path.join(os.path.dirname(_HERE), "include", "spmv.h")

ORIGINAL, RANDOM, RABBIT, RABBITPP, HUBSORT, INSULAR, HUBGROUP, DEGSORT, HUBSORT_ONLY = range(9)
METHODS = {"original": ORIGINAL, "random": RANDOM, "rabbit": RABBIT, "rabbitpp": RABBITPP,
           "hubsort": HUBSORT, "insular": INSULAR, "hubgroup": HUBGROUP, "degsort": DEGSORT,
           "hubsort_only": HUBSORT_ONLY}
STATUS = {0: "SPMV_OK", 1: "SPMV_EINVAL", 2: "SPMV_EPERM", 3: "SPMV_ENOMEM", 4: "SPMV_ECUDA",
          5: "SPMV_ENCCL", 6: "SPMV_EUNSUPPORTED", 7: "SPMV_ESTATE"}


class SpmvError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class _Csr(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64), ("row_ptr32", ctypes.c_void_p),
                ("row_ptr64", ctypes.c_void_p), ("col_idx", ctypes.c_void_p),
                ("vals", ctypes.c_void_p)]


class _Opts(ctypes.Structure):
    _fields_ = [("l2_window", ctypes.c_int32), ("evict_first", ctypes.c_int32),
                ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("device", ctypes.c_int32), ("smem_window", ctypes.c_int32),
                ("l2_hit_ratio", ctypes.c_double), ("variant", ctypes.c_int64),
                ("hot_x", ctypes.c_int64), ("nccl_comm", ctypes.c_void_p),
                ("x_layout", ctypes.c_int32), ("exchange", ctypes.c_int32),
                ("reserved", ctypes.c_int64 * 4)]


XLAYOUT_GLOBAL, XLAYOUT_PADDED = 0, 1
EXCHANGE_COLL, EXCHANGE_PEER = 0, 1

# spmv_coll_t callbacks (int return, 0 = ok)
ALLREDUCE_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64,
                                ctypes.c_void_p)
ALLGATHERV_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                                 ctypes.POINTER(ctypes.c_int64), ctypes.c_int, ctypes.c_void_p)


class _Coll(ctypes.Structure):
    _fields_ = [("ctx", ctypes.c_void_p), ("allreduce_sum_f64", ALLREDUCE_FN),
                ("allgatherv_f32", ALLGATHERV_FN)]


class _Info(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int64) for n in (
        "n", "nnz", "row_begin", "row_end", "nnz_local", "x_len", "x_stride", "y_offset",
        "n_tiles", "n_warp_rows", "n_cta_rows", "n_hub_rows", "n_hub_chunks", "n_mid_rows",
        "hot_prefix", "ideal_bytes")] + \
        [(n, ctypes.c_int32) for n in ("offset_bytes", "world", "rank", "permuted",
                                       "l2_window_bytes", "stream_evict_first", "exec_launches", "spmm4_launches")] + \
        [("hot_prefix_nnz", ctypes.c_int64), ("lane_nnz", ctypes.c_int64),
         ("lane_waste_slots", ctypes.c_int64), ("lane_pred_gather", ctypes.c_int32),
         ("reserved0", ctypes.c_int32)]


class _Stats(ctypes.Structure):
    _fields_ = [("n_communities", ctypes.c_int64), ("largest_comm_frac", ctypes.c_double),
                ("modularity", ctypes.c_double), ("modularity_num", ctypes.c_double),
                ("two_m", ctypes.c_int64), ("n_merges", ctypes.c_int64),
                ("insularity", ctypes.c_double), ("insular_frac", ctypes.c_double),
                ("n_hubs", ctypes.c_int64), ("n_group0", ctypes.c_int64),
                ("skew", ctypes.c_double), ("seconds", ctypes.c_double),
                ("seconds_detect", ctypes.c_double), ("n_deferred", ctypes.c_int64),
                ("parallel", ctypes.c_int32), ("reserved", ctypes.c_int32),
                ("n_insular", ctypes.c_int64)]


_lib = None


def lib() -> ctypes.CDLL:
    """Load libspmv.so (built in-tree by build.py / __graft_entry__.build())."""
    global _lib
    if _lib is None:
        if not os.path.exists(SO_PATH):
            raise ImportError(f"{SO_PATH} is missing: run `python -m paper_conf_ispass_balajicjk23_b200.build`")
        L = ctypes.CDLL(SO_PATH)
        vp, i64, i32, dp = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_void_p
        sig = {
            "spmv_opts_default": (None, [ctypes.POINTER(_Opts)]),
            "spmv_plan": (i32, [ctypes.POINTER(_Csr), vp, ctypes.POINTER(_Opts), ctypes.POINTER(vp)]),
            "spmv_permute": (i32, [vp, vp]),
            "spmv_permute_vec": (i32, [vp, vp, vp, i32, vp]),
            "spmv_pad_vec": (i32, [vp, vp, vp, i32, vp]),
            "spmv_exec": (i32, [vp, vp, vp, vp]),
            "spmv_exec_scaled": (i32, [vp, vp, vp, dp, dp, vp]),
            "spmv_exec_spmm4": (i32, [vp, vp, vp, vp]),
            "spmv_exec_coo": (i32, [vp, vp, vp, vp]),
            "spmv_rabbitpp_gpu": (i32, [ctypes.POINTER(_Csr), vp, vp, vp, vp]),
            "spmv_exec_scaled_bcast": (i32, [vp, vp, vp, i32, dp, dp, vp]),
            "spmv_ipc_handle": (i32, [vp, vp]),
            "spmv_dev_alloc": (i32, [i32, i64, ctypes.POINTER(vp)]),
            "spmv_dev_free": (i32, [vp]),
            "spmv_ipc_open": (i32, [vp, ctypes.POINTER(vp)]),
            "spmv_ipc_close": (i32, [vp]),
            "spmv_export_coo_rows": (i32, [vp, vp, vp]),
            "spmv_iterate": (i32, [vp, vp, i32, ctypes.POINTER(ctypes.c_double), vp]),
            "spmv_scale_vec": (i32, [vp, vp, i64, dp, vp]),
            "spmv_set_coll": (i32, [vp, ctypes.POINTER(_Coll)]),
            "spmv_set_peers": (i32, [vp, vp, i32]),
            "spmv_iterate_finish": (i32, [vp, vp, i64, dp, ctypes.POINTER(ctypes.c_double), vp]),
            "spmv_plan_info": (i32, [vp, ctypes.POINTER(_Info)]),
            "spmv_export_csr": (i32, [vp, vp, vp, vp, vp]),
            "spmv_export_bins": (i32, [vp, vp, vp, vp, vp, vp, vp, vp, vp]),
            "spmv_export_partition": (i32, [vp, vp]),
            "spmv_export_inverse": (i32, [vp, vp, vp]),
            "spmv_destroy": (None, [vp]),
            "spmv_reset_persisting_l2": (i32, [vp]),
            "spmv_reorder": (i32, [i64, i64, vp, vp, i32, ctypes.c_uint64, vp, ctypes.POINTER(_Stats)]),
            "spmv_reorder_last_comm": (i32, [i64, vp]),
            "spmv_reorder_last_merges": (i32, [i64, vp, vp, vp, ctypes.POINTER(ctypes.c_int64)]),
            "spmv_last_error": (ctypes.c_char_p, []),
            "spmv_version": (ctypes.c_char_p, []),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def declared_symbols() -> list[str]:
    """Every function include/spmv.h declares."""
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"^\s*(?:spmv_status|void|const char\*)\s+(spmv_\w+)\s*\(", txt, re.M)))


def _check(st: int):
    if st != 0:
        raise SpmvError(st, lib().spmv_last_error().decode())


def version() -> str:
    return lib().spmv_version().decode()


def _stream_ptr(stream=None, device=None) -> int:
    """The given stream, else the current stream of `device` (a plan's device,
    not whichever device happens to be current)."""
    import torch
    s = stream if stream is not None else torch.cuda.current_stream(device)
    return int(s.cuda_stream)


def _ptr(t) -> int | None:
    return None if t is None else int(t.data_ptr())


class Plan:
    """spmv_plan + spmv_permute over device CSR tensors (torch, cuda).

    row_ptr: int32 or int64 [n+1]; col: int32 [nnz]; val: float32 [nnz];
    perm: int32 [n] (perm[old] = new) or None for identity.
    """

    def __init__(self, row_ptr, col, val, perm=None, *, world=1, rank=0, l2_window=True,
                 evict_first=True, l2_hit_ratio=1.0, smem_window=True, variant=0,
                 hot_x=0, permute=True, stream=None, x_layout=XLAYOUT_GLOBAL,
                 exchange=EXCHANGE_COLL, nccl_comm=None):
        import torch
        assert row_ptr.is_cuda and col.is_cuda and val.is_cuda
        assert col.dtype == torch.int32 and val.dtype == torch.float32
        n = row_ptr.numel() - 1
        self._keep = (row_ptr, col, val, perm)  # A must outlive permute
        A = _Csr(n, col.numel(), None, None, _ptr(col), _ptr(val))
        if row_ptr.dtype == torch.int64:
            A.row_ptr64 = _ptr(row_ptr)
        elif row_ptr.dtype == torch.int32:
            A.row_ptr32 = _ptr(row_ptr)
        else:
            raise TypeError("row_ptr must be int32 or int64")
        if perm is not None:
            assert perm.is_cuda and perm.dtype == torch.int32 and perm.numel() == n
        o = _Opts()
        lib().spmv_opts_default(ctypes.byref(o))
        o.world, o.rank = world, rank
        o.l2_window, o.evict_first = int(l2_window), int(evict_first)
        o.l2_hit_ratio = l2_hit_ratio
        o.smem_window = int(smem_window)
        o.variant = int(variant)
        o.hot_x = int(hot_x)
        o.x_layout, o.exchange = int(x_layout), int(exchange)
        o.nccl_comm = nccl_comm
        o.device = row_ptr.device.index if row_ptr.device.index is not None else -1
        h = ctypes.c_void_p()
        _check(lib().spmv_plan(ctypes.byref(A), _ptr(perm), ctypes.byref(o), ctypes.byref(h)))
        self._h = h
        self.device = row_ptr.device
        if permute:
            self.permute(stream)

    # ------------------------------------------------------------------ calls
    def permute(self, stream=None):
        _check(lib().spmv_permute(self._h, _stream_ptr(stream, self.device)))
        return self

    def info(self) -> dict:
        i = _Info()
        _check(lib().spmv_plan_info(self._h, ctypes.byref(i)))
        return {f: getattr(i, f) for f, _ in _Info._fields_ if f not in ("r0", "r1", "r2")}

    def permute_vec(self, x, inverse=False, out=None, stream=None):
        import torch
        out = torch.empty_like(x) if out is None else out
        _check(lib().spmv_permute_vec(self._h, _ptr(x), _ptr(out), int(inverse), _stream_ptr(stream, self.device)))
        return out

    def pad_vec(self, x, to_padded=True, out=None, stream=None):
        import torch
        if out is None:
            info = self.info()
            out = torch.zeros(info["x_len"] if to_padded else info["n"], dtype=torch.float32,
                              device=x.device)
        _check(lib().spmv_pad_vec(self._h, _ptr(x), _ptr(out), int(to_padded), _stream_ptr(stream, self.device)))
        return out

    def exec(self, x, y=None, stream=None):
        import torch
        if y is None:
            info = self.info()
            y = torch.empty(info["row_end"] - info["row_begin"], dtype=torch.float32, device=x.device)
        _check(lib().spmv_exec(self._h, _ptr(x), _ptr(y), _stream_ptr(stream, self.device)))
        return y

    def exec_coo(self, x, y=None, stream=None):
        """y_B = B x_B reading B as COO triplets (SpMV-COO)."""
        import torch
        if y is None:
            info = self.info()
            y = torch.empty(info["row_end"] - info["row_begin"], dtype=torch.float32, device=x.device)
        _check(lib().spmv_exec_coo(self._h, _ptr(x), _ptr(y), _stream_ptr(stream, self.device)))
        return y

    def export_coo_rows(self):
        import torch
        info = self.info()
        rows = torch.empty(info["nnz_local"], dtype=torch.int32, device=self.device)
        _check(lib().spmv_export_coo_rows(self._h, _ptr(rows), _stream_ptr(None, self.device)))
        return rows

    def exec_spmm4(self, X, Y=None, stream=None):
        """Y_B = B X_B for X_B of shape (x_len, 4), row-major fp32 (SpMM-CSR-4)."""
        import torch
        if Y is None:
            info = self.info()
            Y = torch.empty((info["row_end"] - info["row_begin"], 4), dtype=torch.float32,
                            device=X.device)
        _check(lib().spmv_exec_spmm4(self._h, _ptr(X), _ptr(Y), _stream_ptr(stream, self.device)))
        return Y

    def exec_scaled_bcast(self, x, x_next_ptrs, sumsq_in, sumsq_out, stream=None):
        """Fused exec + exchange: rows scaled as exec_scaled, stored into every
        buffer of x_next_ptrs (device addresses, padded x layout)."""
        arr = (ctypes.c_void_p * len(x_next_ptrs))(*[int(a) for a in x_next_ptrs])
        _check(lib().spmv_exec_scaled_bcast(self._h, _ptr(x), arr, len(x_next_ptrs),
                                            _ptr(sumsq_in), _ptr(sumsq_out), _stream_ptr(stream, self.device)))

    def exec_scaled(self, x, y, sumsq_in=None, sumsq_out=None, stream=None):
        _check(lib().spmv_exec_scaled(self._h, _ptr(x), _ptr(y), _ptr(sumsq_in), _ptr(sumsq_out),
                                      _stream_ptr(stream, self.device)))
        return y

    def set_coll(self, coll):
        """Install a collective backend (a _Coll, kept alive here) or None for
        NCCL on the plan's nccl_comm."""
        self._coll = coll
        _check(lib().spmv_set_coll(self._h, None if coll is None else ctypes.byref(coll)))

    def set_peers(self, ptrs):
        """Peer next-x buffers of the PEER exchange: 2 * world device addresses,
        [j * world + k] = buffer j of rank k."""
        arr = (ctypes.c_void_p * len(ptrs))(*ptrs)
        _check(lib().spmv_set_peers(self._h, ctypes.cast(arr, ctypes.c_void_p),
                                    len(ptrs) // 2))

    def iterate(self, x, iters: int, stream=None) -> float:
        lam = ctypes.c_double(0.0)
        _check(lib().spmv_iterate(self._h, _ptr(x), iters, ctypes.byref(lam), _stream_ptr(stream, self.device)))
        return lam.value

    def export_csr(self, stream=None):
        import torch
        i = self.info()
        nr = i["row_end"] - i["row_begin"]
        rp = torch.empty(nr + 1, dtype=torch.int64, device=self.device)
        col = torch.empty(max(i["nnz_local"], 0), dtype=torch.int32, device=self.device)
        val = torch.empty(max(i["nnz_local"], 0), dtype=torch.float32, device=self.device)
        _check(lib().spmv_export_csr(self._h, _ptr(rp), _ptr(col), _ptr(val), _stream_ptr(stream, self.device)))
        return rp, col, val

    def export_bins(self, stream=None) -> dict:
        import torch
        i = self.info()
        mk = lambda m: torch.empty(max(m, 0), dtype=torch.int32, device=self.device)  # noqa: E731
        d = {"tiles": mk(i["n_tiles"] + 1), "mid_rows": mk(i["n_mid_rows"]),
             "warp_rows": mk(i["n_warp_rows"]),
             "cta_rows": mk(i["n_cta_rows"]),
             "hub_rows": mk(i["n_hub_rows"]), "chunk_row": mk(i["n_hub_chunks"]),
             "chunk_idx": mk(i["n_hub_chunks"])}
        _check(lib().spmv_export_bins(self._h, _ptr(d["tiles"]), _ptr(d["mid_rows"]),
                                      _ptr(d["warp_rows"]),
                                      _ptr(d["cta_rows"]),
                                      _ptr(d["hub_rows"]), _ptr(d["chunk_row"]),
                                      _ptr(d["chunk_idx"]), _stream_ptr(stream, self.device)))
        return d

    def export_partition(self) -> list[int]:
        w = self.info()["world"]
        b = (ctypes.c_int64 * (w + 1))()
        _check(lib().spmv_export_partition(self._h, ctypes.cast(b, ctypes.c_void_p)))
        return list(b)

    def export_inverse(self, stream=None):
        import torch
        inv = torch.empty(self.info()["n"], dtype=torch.int32, device=self.device)
        _check(lib().spmv_export_inverse(self._h, _ptr(inv), _stream_ptr(stream, self.device)))
        return inv

    def close(self):
        if getattr(self, "_h", None):
            import torch
            torch.cuda.synchronize(self.device)
            lib().spmv_destroy(self._h)
            self._h = None
            self._keep = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def iterate_finish(u, x, sumsq, stream=None) -> float:
    """x = u / sqrt(sumsq) (device), returns lambda = sqrt(sumsq)."""
    lam = ctypes.c_double(0.0)
    _check(lib().spmv_iterate_finish(_ptr(u), _ptr(x), u.numel(), _ptr(sumsq), ctypes.byref(lam),
                                     _stream_ptr(stream, u.device)))
    return lam.value


def scale_vec(u, x, sumsq=None, stream=None):
    _check(lib().spmv_scale_vec(_ptr(u), _ptr(x), u.numel(), _ptr(sumsq), _stream_ptr(stream)))
    return x


@dataclass
class ReorderStats:
    n_communities: int
    largest_comm_frac: float
    modularity: float
    modularity_num: float
    two_m: int
    n_merges: int
    insularity: float
    insular_frac: float
    n_hubs: int
    n_group0: int
    skew: float
    seconds: float
    seconds_detect: float
    n_deferred: int = 0
    parallel: int = 0
    reserved: int = 0
    n_insular: int = 0


PARALLEL, LOG = 0x100, 0x200


def reorder(row_ptr: np.ndarray, col: np.ndarray, method="rabbitpp", seed: int = 0,
            parallel: bool = False, log: bool = False):
    """Host reordering (spmv_reorder).  Returns (perm int32[n], ReorderStats).
    parallel: concurrent RABBIT merges (SPMV_REORDER_PARALLEL); log: keep the
    merge log for reorder_last_merges()."""
    m = METHODS[method] if isinstance(method, str) else int(method)
    m |= (PARALLEL if parallel else 0) | (LOG if log else 0)
    rp = np.ascontiguousarray(row_ptr, dtype=np.int64)
    c = np.ascontiguousarray(col, dtype=np.int32)
    n = len(rp) - 1
    perm = np.empty(n, np.int32)
    st = _Stats()
    _check(lib().spmv_reorder(n, int(rp[-1]) if n >= 0 else 0, rp.ctypes.data, c.ctypes.data, m,
                              seed, perm.ctypes.data, ctypes.byref(st)))
    return perm, ReorderStats(**{f: getattr(st, f) for f, _ in _Stats._fields_})


def reorder_last_merges():
    """(child int32[], root int32[], dq int64[]) of the last logged detection."""
    cnt = ctypes.c_int64(0)
    _check(lib().spmv_reorder_last_merges(0, None, None, None, ctypes.byref(cnt)))
    m = cnt.value
    c, p, d = np.empty(m, np.int32), np.empty(m, np.int32), np.empty(m, np.int64)
    _check(lib().spmv_reorder_last_merges(m, c.ctypes.data, p.ctypes.data, d.ctypes.data,
                                          ctypes.byref(cnt)))
    return c, p, d


def reorder_last_comm(n: int) -> np.ndarray:
    out = np.empty(n, np.int32)
    _check(lib().spmv_reorder_last_comm(n, out.ctypes.data))
    return out


class DeviceBuffer:
    """fp32 device buffer from spmv_dev_alloc (a standalone cudaMalloc, so its
    CUDA IPC handle names exactly this buffer); .tensor views it as torch."""

    def __init__(self, n: int, device: int):
        import torch
        p = ctypes.c_void_p()
        _check(lib().spmv_dev_alloc(int(device), 4 * int(n), ctypes.byref(p)))
        self.ptr, self.n = int(p.value), int(n)
        self.__cuda_array_interface__ = {"shape": (self.n,), "typestr": "<f4",
                                         "data": (self.ptr, False), "version": 3}
        self.tensor = torch.as_tensor(self, device=torch.device("cuda", int(device)))

    def handle(self) -> bytes:
        buf = ctypes.create_string_buffer(64)
        _check(lib().spmv_ipc_handle(ctypes.c_void_p(self.ptr), buf))
        return buf.raw

    def close(self):
        if self.ptr:
            self.tensor = None
            lib().spmv_dev_free(ctypes.c_void_p(self.ptr))
            self.ptr = 0


def ipc_open(handle: bytes) -> int:
    p = ctypes.c_void_p()
    _check(lib().spmv_ipc_open(ctypes.create_string_buffer(handle, 64), ctypes.byref(p)))
    return int(p.value)


def ipc_close(ptr: int) -> None:
    _check(lib().spmv_ipc_close(ctypes.c_void_p(ptr)))


def rabbitpp_gpu(row_ptr, col, perm_rabbit, comm, stream=None):
    """RABBIT++ post-pass on the GPU (spmv_rabbitpp_gpu): device tensors in,
    device int32 permutation out."""
    import torch
    n = row_ptr.numel() - 1
    A = _Csr(n, col.numel(), None, None, _ptr(col), None)
    if row_ptr.dtype == torch.int64:
        A.row_ptr64 = _ptr(row_ptr)
    else:
        A.row_ptr32 = _ptr(row_ptr)
    out = torch.empty(n, dtype=torch.int32, device=col.device)
    _check(lib().spmv_rabbitpp_gpu(ctypes.byref(A), _ptr(perm_rabbit), _ptr(comm), _ptr(out),
                                   _stream_ptr(stream)))
    return out
