"""B200-native SpMV hot path of the PEPPHER composition tool (Dastgeer, Li,
Kessler, MuCoCoS 2012): y = A·x over CSR in fp64, three hand-written sm_100a
variants, per-call history-based variant selection, nnz-balanced row
partitioning over ranks with NCCL exchange.

This module is the thin Python binding of ``include/pepp_spmv.h``: it only
marshals arguments (pointers, sizes, the caller's CUDA stream) into
``libpepp_spmv.so``. Every step of the path runs in that library's kernels.
Device memory, streams and process groups come from PyTorch (plumbing).
There is no CPU fallback: importing works without a GPU, but planning needs
the CUDA library and a device and fails loudly otherwise.
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass
from typing import Optional, Sequence

import numpy as np

from . import _capi as C
from ._capi import (ACCESS_READ, ACCESS_READWRITE, ACCESS_WRITE, DEVICE_SIMULATED, EXEC_NO_TIMING, PeppError, V_CSR_STREAM, V_CSR_VECTOR, V_MERGE_PATH, V_PANEL, V_SELL, X_ALLGATHER, X_AUTO,
                    X_HALO, X_NONE, X_P2P, Y_LOCAL, Y_NEXT_INPUT, Y_REPLICATED, VARIANT_NAMES)

__all__ = ["Plan", "Choice", "History", "Vector", "ACCESS_READ", "ACCESS_WRITE", "ACCESS_READWRITE",
           "DEVICE_SIMULATED", "partition_rows", "halo_ghosts", "context_key", "nccl_unique_id", "dist_choose",
           "lib_path", "PeppError", "V_CSR_VECTOR", "V_MERGE_PATH", "V_SELL", "V_CSR_STREAM", "V_PANEL", "X_AUTO", "X_NONE",
           "X_ALLGATHER", "X_HALO", "X_P2P", "Y_LOCAL", "Y_NEXT_INPUT", "Y_REPLICATED", "EXEC_NO_TIMING",
           "VARIANT_NAMES"]

lib_path = C.LIB_PATH


@dataclass(slots=True)
class Choice:
    variant: int
    param: int = 0
    exchange: int = X_AUTO
    nparts: int = 0          # force: 0 = this rank's own block (P' = nranks); P' < nranks = a distribution
    calibrating: bool = False
    candidate: int = -1
    predicted_us: float = 0.0
    launches: int = 0
    layout_bytes: int = 0

    @property
    def name(self) -> str:
        return f"{VARIANT_NAMES.get(self.variant, self.variant)}[{self.param}]"

    @staticmethod
    def _from(c: C.CHOICE_T) -> "Choice":
        return Choice(c.variant, c.param, c.exchange, c.nparts, bool(c.calibrating), c.candidate, c.predicted_us,
                      c.launches, c.layout_bytes)

    def _to(self) -> C.CHOICE_T:
        c = C.CHOICE_T()
        c.variant, c.param, c.exchange, c.nparts = self.variant, self.param, self.exchange, self.nparts
        return c


def _ptr(a) -> int:
    """Raw address of a numpy array or torch tensor (no copy)."""
    if a is None:
        return 0
    if isinstance(a, np.ndarray):
        return a.ctypes.data
    return int(a.data_ptr())


def _stream_handle(stream) -> int:
    if stream is None:
        import torch
        if not torch.cuda.is_available():
            return 0   # legacy default stream (the library reports PEPP_E_CUDA where a device is needed)
        raw = getattr(torch._C, "_cuda_getCurrentRawStream", None)   # torch's current stream, without a Stream object
        if raw is not None:
            return int(raw(torch._C._cuda_getDevice()))
        return int(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return stream
    return int(stream.cuda_stream)


class Plan:
    """pepp_spmv_plan over one CSR row block.

    ``row_ptr`` (int64, global offsets: row_ptr[0] == first), ``col`` (int32),
    ``val`` (float64, or float32 for the fp32 instance — the value type of
    the plan, and of every x / y passed to it): numpy host arrays, or CUDA
    torch tensors on the plan's device (then ``on_device`` is inferred). The
    plan copies them.
    """

    def __init__(self, nrows: int, ncols: int, row_ptr, col, val, *, variant_mask: Optional[int] = None,
                 use_history: Optional[bool] = None, validate: bool = True, sell_sigma: int = 0,
                 device: Optional[int] = None, min_samples: int = 3, sample_period: int = 8,
                 nranks: int = 1, rank: int = 0, row_bounds: Optional[Sequence[int]] = None,
                 nccl_unique_id: Optional[bytes] = None, exchange: int = X_AUTO,
                 history_path: Optional[str] = None, prune: bool = True, overlap: bool = True,
                 predict=None, compress_values: bool = True, dist_select: bool = True):
        L = C.lib()
        self._h = ctypes.c_void_p()
        on_dev = not isinstance(row_ptr, np.ndarray)
        if not on_dev:
            f32 = np.asarray(val).dtype == np.float32
            row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
            col = np.ascontiguousarray(col, dtype=np.int32)
            val = np.ascontiguousarray(val, dtype=np.float32 if f32 else np.float64)
        else:
            import torch
            f32 = val.dtype == torch.float32
        nnz = int(col.shape[0]) if col is not None else 0
        first = int(row_ptr[0]) if not on_dev else int(row_ptr[:1].cpu()[0])
        self.value_type = C.VALUE_F32 if f32 else C.VALUE_F64
        A = C.CSR_T(nrows, ncols, nnz, first, _ptr(row_ptr), _ptr(col) if nnz else 0,
                    _ptr(val) if nnz else 0, 1 if on_dev else 0, self.value_type)
        o = C.OPTS_T()
        L.pepp_spmv_opts_default(ctypes.byref(o))
        # None keeps pepp_spmv_opts_default's value (which honours the global
        # switches PEPP_VARIANT / PEPP_USE_HISTORY / PEPP_HISTORY_PATH)
        if variant_mask is not None:
            o.variant_mask = variant_mask
        if use_history is not None:
            o.use_history = 1 if use_history else 0
        o.validate = 1 if validate else 0
        o.sell_sigma = sell_sigma
        o.device = -1 if device is None else device
        o.min_samples = min_samples
        o.sample_period = sample_period
        o.nranks, o.rank = nranks, rank
        self._bounds = None
        if row_bounds is not None:
            self._bounds = np.ascontiguousarray(row_bounds, dtype=np.int64)
            o.row_bounds = self._bounds.ctypes.data
        self._uid = None
        if nccl_unique_id is not None:
            self._uid = ctypes.create_string_buffer(bytes(nccl_unique_id), 128)
            o.nccl_unique_id = ctypes.addressof(self._uid)
        o.exchange = exchange
        self._hp = history_path.encode() if history_path else None
        if self._hp is not None:
            o.history_path = self._hp
        o.prune = 1 if prune else 0
        o.overlap = 1 if overlap else 0
        o.compress_values = 1 if compress_values else 0
        o.dist_select = 1 if dist_select else 0
        cb = None
        if predict is not None:
            # predict(context: dict, variant: int, param: int) -> µs (<= 0: no prediction);
            # called only inside pepp_spmv_plan (the descriptor's prediction function, P@6887)
            def _cb(info_p, variant, param, _user):
                try:
                    return float(predict(info_p.contents.as_dict(), int(variant), int(param)))
                except Exception:   # never unwind through the C caller
                    return -1.0
            cb = C.PREDICT_FN(_cb)
            o.predict = cb
        C.check(L.pepp_spmv_plan(ctypes.byref(A), ctypes.byref(o), ctypes.byref(self._h)), "pepp_spmv_plan")
        self.nrows, self.ncols, self.nnz = nrows, ncols, nnz
        self._global_rows = int(self._bounds[-1]) if self._bounds is not None else nrows
        # per-call fast path of exec: the bound C function, a reused result struct,
        # the torch dtype of the plan's value type (None without torch)
        self._fexec = L.pepp_spmv_exec
        self._used = C.CHOICE_T()
        self._used_ref = ctypes.byref(self._used)
        try:
            import torch
            self._tdtype = torch.float32 if f32 else torch.float64
        except ImportError:
            self._tdtype = None

    # ---- calls ----
    def _vec(self, t, n: int, name: str) -> int:
        """Device address of an operand: a contiguous CUDA tensor of the plan's
        value type with at least `n` entries, or a raw device address (int,
        unchecked). Host arrays are refused (exec_host takes those): the C
        entry points get plain pointers and cannot tell."""
        td = self._tdtype
        if td is not None and getattr(t, "dtype", None) is td and t.is_cuda and t.is_contiguous() and t.numel() >= n:
            return t.data_ptr()   # the common case, checked cheaply
        if t is None or isinstance(t, int):
            return t or 0
        if isinstance(t, np.ndarray):
            raise TypeError(f"{name}: a host array; pass a CUDA tensor (or use exec_host / exec_host_batch)")
        want = "float32" if self.value_type == C.VALUE_F32 else "float64"
        if not getattr(t, "is_cuda", False) or str(t.dtype).rpartition(".")[2] != want:
            raise TypeError(f"{name}: expected a CUDA {want} tensor, got {getattr(t, 'device', '?')} {t.dtype}")
        if not t.is_contiguous() or t.numel() < n:
            raise ValueError(f"{name}: needs a contiguous tensor of >= {n} entries, got {tuple(t.shape)}")
        return int(t.data_ptr())

    def exec(self, x, y, flags: int = Y_LOCAL, stream=None, force: Optional[Choice] = None) -> Choice:
        """y = A·x (x: ncols entries, y: global rows; CUDA tensors of the plan's
        value type). Asynchronous on ``stream``."""
        f = ctypes.byref(force._to()) if force is not None else None
        px, py = self._vec(x, self.ncols, "x"), self._vec(y, self._global_rows, "y")
        st = stream.cuda_stream if hasattr(stream, "cuda_stream") else _stream_handle(stream)
        r = self._fexec(self._h, px, py, flags, st, f, self._used_ref)
        if r:
            C.check(r, "pepp_spmv_exec")
        return Choice._from(self._used)

    def exec_vec(self, x: "Vector", y: "Vector", flags: int = Y_LOCAL, stream=None,
                 force: Optional[Choice] = None) -> Choice:
        """y = A·x through smart containers (x READ, y WRITE); copies only what the states require."""
        used = C.CHOICE_T()
        f = force._to() if force is not None else None
        C.check(C.lib().pepp_spmv_exec_vec(self._h, x._h, y._h, flags, _stream_handle(stream),
                                           ctypes.byref(f) if f is not None else None, ctypes.byref(used)),
                "pepp_spmv_exec_vec")
        return Choice._from(used)

    def graph(self, x, y, iterations: int = 1, mode: int = 0, work=None, flags: int = Y_LOCAL,
              stream=None) -> "Graph":
        """Capture `iterations` calls into a CUDA graph (mode 0: repeat y = A·x;
        mode 1: iterate, ping-pong y / work)."""
        g = ctypes.c_void_p()
        px, py = self._vec(x, self.ncols, "x"), self._vec(y, self._global_rows, "y")
        pw = self._vec(work, self._global_rows, "work")
        C.check(C.lib().pepp_spmv_graph_create(self._h, px, py, pw, iterations, mode, flags,
                                               _stream_handle(stream), ctypes.byref(g)), "pepp_spmv_graph_create")
        return Graph(g, (x, y, work))

    def exchange(self, y, flags: int = Y_NEXT_INPUT, stream=None) -> None:
        """The exchange step alone (no-op on an unpartitioned plan)."""
        C.check(C.lib().pepp_spmv_exchange(self._h, self._vec(y, self._global_rows, "y"), flags, _stream_handle(stream)),
                "pepp_spmv_exchange")

    def p2p_buffers(self, nbuf: int = 2) -> list:
        """pepp_spmv_p2p_buffers (collective): `nbuf` plan-owned symmetric
        device buffers (global length, the plan's value type) as CUDA tensors.
        PEPP_Y_NEXT_INPUT calls whose y is one of them push the halo from the
        boundary kernel straight into the peers' copies (PEPP_X_P2P). The
        tensors borrow the plan's memory: they keep the Plan object alive, and
        must not be used after close()."""
        import torch
        arr = (ctypes.c_void_p * nbuf)()
        C.check(C.lib().pepp_spmv_p2p_buffers(self._h, nbuf, arr), "pepp_spmv_p2p_buffers")
        n = int(self._bounds[-1]) if self._bounds is not None else self.nrows
        f32 = self.value_type == C.VALUE_F32
        dev = torch.cuda.current_device()
        out = []
        for i in range(nbuf):
            ref = _DeviceArray(arr[i], n, "<f4" if f32 else "<f8", self)
            out.append(torch.as_tensor(ref, device=torch.device("cuda", dev)))
        return out

    def exec_host(self, x_host: np.ndarray, y_host: np.ndarray, iterations: int = 1, flags: int = Y_LOCAL,
                  stream=None) -> None:
        """Host buffers in and out, transfers inside the call (synchronous)."""
        want = np.float32 if self.value_type == C.VALUE_F32 else np.float64
        for a, n, name in ((x_host, self.ncols, "x_host"), (y_host, self._global_rows, "y_host")):
            if not isinstance(a, np.ndarray) or a.dtype != want or not a.flags.c_contiguous or a.size < n:
                raise ValueError(f"{name}: needs a contiguous {np.dtype(want).name} array of >= {n} entries")
        C.check(C.lib().pepp_spmv_exec_host(self._h, _ptr(x_host), _ptr(y_host), iterations, flags,
                                            _stream_handle(stream)), "pepp_spmv_exec_host")

    def exec_host_batch(self, x_hosts: Sequence[np.ndarray], y_hosts: Sequence[np.ndarray], iterations: int = 1,
                        flags: int = Y_LOCAL, stream=None) -> None:
        """exec_host over independent right-hand sides, transfers overlapped
        with the computation (synchronous)."""
        want = np.float32 if self.value_type == C.VALUE_F32 else np.float64
        if len(x_hosts) != len(y_hosts):
            raise ValueError("x_hosts and y_hosts differ in length")
        for arrs, n, name in ((x_hosts, self.ncols, "x_hosts"), (y_hosts, self._global_rows, "y_hosts")):
            for a in arrs:
                if not isinstance(a, np.ndarray) or a.dtype != want or not a.flags.c_contiguous or a.size < n:
                    raise ValueError(f"{name}: needs contiguous {np.dtype(want).name} arrays of >= {n} entries")
        n = len(x_hosts)
        xs = (ctypes.c_void_p * max(n, 1))(*[_ptr(a) for a in x_hosts])
        ys = (ctypes.c_void_p * max(n, 1))(*[_ptr(a) for a in y_hosts])
        C.check(C.lib().pepp_spmv_exec_host_batch(self._h, n, xs, ys, iterations, flags, _stream_handle(stream)),
                "pepp_spmv_exec_host_batch")

    def select(self) -> Choice:
        c = C.CHOICE_T()
        C.check(C.lib().pepp_spmv_select(self._h, ctypes.byref(c)), "pepp_spmv_select")
        return Choice._from(c)

    def candidates(self) -> list[Choice]:
        n = ctypes.c_int32()
        C.check(C.lib().pepp_spmv_candidates(self._h, None, 0, ctypes.byref(n)), "pepp_spmv_candidates")
        arr = (C.CHOICE_T * max(1, n.value))()
        C.check(C.lib().pepp_spmv_candidates(self._h, arr, n.value, ctypes.byref(n)), "pepp_spmv_candidates")
        return [Choice._from(arr[i]) for i in range(n.value)]

    def info(self) -> dict:
        i = C.INFO_T()
        C.check(C.lib().pepp_spmv_plan_info(self._h, ctypes.byref(i)), "pepp_spmv_plan_info")
        return i.as_dict()

    def dist_stats(self) -> list[tuple[int, int, float]]:
        """(P', exchange, agreed mean µs) per distribution candidate (opts.dist_select)."""
        n = ctypes.c_int32()
        C.check(C.lib().pepp_spmv_dist_stats(self._h, 0, None, None, None, ctypes.byref(n)), "pepp_spmv_dist_stats")
        k = max(1, n.value)
        pa, ex, us = np.zeros(k, np.int32), np.zeros(k, np.int32), np.zeros(k, np.float64)
        C.check(C.lib().pepp_spmv_dist_stats(self._h, k, pa.ctypes.data, ex.ctypes.data, us.ctypes.data,
                                             ctypes.byref(n)), "pepp_spmv_dist_stats")
        return [(int(pa[i]), int(ex[i]), float(us[i])) for i in range(n.value)]

    def flush_history(self) -> None:
        C.check(C.lib().pepp_spmv_flush_history(self._h), "pepp_spmv_flush_history")

    def history_stats(self, cand: int) -> tuple[int, float, float]:
        n, m, m2 = ctypes.c_int64(), ctypes.c_double(), ctypes.c_double()
        C.check(C.lib().pepp_spmv_history_stats(self._h, cand, ctypes.byref(n), ctypes.byref(m), ctypes.byref(m2)),
                "pepp_spmv_history_stats")
        return n.value, m.value, m2.value

    def close(self) -> None:
        if getattr(self, "_h", None) and self._h.value:
            C.check(C.lib().pepp_spmv_destroy(self._h), "pepp_spmv_destroy")
            self._h = ctypes.c_void_p()

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @classmethod
    def from_csr(cls, A, **kw) -> "Plan":
        """From any object with nrows, ncols, row_ptr, col, val (e.g. gen.CSR)."""
        return cls(A.nrows, A.ncols, A.row_ptr, A.col, A.val, **kw)


class _DeviceArray:
    """__cuda_array_interface__ view of plan-owned device memory (no copy);
    holds the plan so the memory outlives every tensor made from it."""

    def __init__(self, ptr: int, n: int, typestr: str, owner):
        self._owner = owner
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (int(ptr), False),
                                         "version": 3, "strides": None}


class Graph:
    """A captured sequence of SpMV calls (pepp_spmv_graph_*)."""

    def __init__(self, h, keep):
        self._h = h
        self._keep = keep   # the buffers the graph reads / writes must stay alive

    def launch(self, stream=None) -> None:
        C.check(C.lib().pepp_spmv_graph_launch(self._h, _stream_handle(stream)), "pepp_spmv_graph_launch")

    def close(self) -> None:
        if self._h and self._h.value:
            C.lib().pepp_spmv_graph_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Vector:
    """Smart container for one fp64 vector (pepp_vector_*): a host master copy
    plus a lazily allocated device copy with valid / outdated states
    (paper §IV-D, Fig. 3). ``host`` (numpy float64) is borrowed as the master
    copy, or one is allocated (pinned)."""

    def __init__(self, n: int, host: Optional[np.ndarray] = None, device: Optional[int] = None):
        self._h = ctypes.c_void_p()
        self._host_ref = None
        hp = 0
        if host is not None:
            assert host.dtype == np.float64 and host.flags.c_contiguous and host.size == n
            self._host_ref = host
            hp = host.ctypes.data
        C.check(C.lib().pepp_vector_create(n, hp or None, -1 if device is None else device, ctypes.byref(self._h)),
                "pepp_vector_create")
        self.n = n

    def host(self, mode: int = ACCESS_READ) -> np.ndarray:
        """Host access with `mode`: returns the (now valid) master copy as a numpy view."""
        p = ctypes.c_void_p()
        C.check(C.lib().pepp_vector_acquire_host(self._h, mode, ctypes.byref(p)), "pepp_vector_acquire_host")
        if self._host_ref is not None:
            return self._host_ref
        return np.ctypeslib.as_array(ctypes.cast(p, ctypes.POINTER(ctypes.c_double)), shape=(self.n,))

    def device(self, mode: int, stream=None) -> int:
        """Device access with `mode` (copy enqueued if needed); returns the device pointer."""
        p = ctypes.c_void_p()
        C.check(C.lib().pepp_vector_acquire_device(self._h, mode, _stream_handle(stream) if stream is not False else None,
                                                   ctypes.byref(p)), "pepp_vector_acquire_device")
        return p.value or 0

    def release(self, stream=None) -> None:
        C.check(C.lib().pepp_vector_release_device(self._h, _stream_handle(stream) if stream is not False else None),
                "pepp_vector_release_device")

    def scale(self, alpha: float, stream=None) -> None:
        """A READWRITE component: v = alpha * v on the device."""
        C.check(C.lib().pepp_vector_scale(self._h, alpha, _stream_handle(stream) if stream is not False else None),
                "pepp_vector_scale")

    def counters(self) -> tuple[int, int, int]:
        a, b, c = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        C.check(C.lib().pepp_vector_counters(self._h, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c)),
                "pepp_vector_counters")
        return a.value, b.value, c.value

    def state(self) -> tuple[bool, bool]:
        h, d = ctypes.c_int32(), ctypes.c_int32()
        C.check(C.lib().pepp_vector_state(self._h, ctypes.byref(h), ctypes.byref(d)), "pepp_vector_state")
        return bool(h.value), bool(d.value)

    def close(self) -> None:
        if getattr(self, "_h", None) and self._h.value:
            C.lib().pepp_vector_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class History:
    """Stand-alone history table + selection policy (host only; see header)."""

    def __init__(self):
        self._h = ctypes.c_void_p()
        C.check(C.lib().pepp_history_create(ctypes.byref(self._h)), "pepp_history_create")

    def record(self, key: int, cand: int, us: float) -> None:
        C.check(C.lib().pepp_history_record(self._h, key, cand, us), "pepp_history_record")

    def stats(self, key: int, cand: int) -> tuple[int, float, float]:
        n, m, m2 = ctypes.c_int64(), ctypes.c_double(), ctypes.c_double()
        C.check(C.lib().pepp_history_stats(self._h, key, cand, ctypes.byref(n), ctypes.byref(m), ctypes.byref(m2)),
                "pepp_history_stats")
        return n.value, m.value, m2.value

    def select(self, key: int, eligible: Sequence[bool], min_samples: int = 3) -> tuple[int, bool, float]:
        e = np.ascontiguousarray([1 if v else 0 for v in eligible], dtype=np.uint8)
        c, cal, pred = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_double()
        C.check(C.lib().pepp_history_select(self._h, key, len(e), e.ctypes.data, min_samples, ctypes.byref(c),
                                            ctypes.byref(cal), ctypes.byref(pred)), "pepp_history_select")
        return c.value, bool(cal.value), pred.value

    def prior(self, key: int, ids: Sequence[int]):
        """(prior means per id or -1, source key) from the nearest recorded context, or None."""
        a = np.ascontiguousarray(ids, dtype=np.int32)
        out = np.empty(len(a), dtype=np.float64)
        k = ctypes.c_uint64()
        st = C.lib().pepp_history_prior(self._h, key, len(a), a.ctypes.data, out.ctypes.data, ctypes.byref(k))
        if st == C.PEPP_E_STATE:
            return None
        C.check(st, "pepp_history_prior")
        return out, k.value

    def save(self, path: str) -> None:
        C.check(C.lib().pepp_history_save(self._h, path.encode()), "pepp_history_save")

    def load(self, path: str) -> None:
        C.check(C.lib().pepp_history_load(self._h, path.encode()), "pepp_history_load")

    def close(self) -> None:
        if self._h.value:
            C.lib().pepp_history_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def partition_rows(row_ptr: np.ndarray, nparts: int) -> np.ndarray:
    """nnz-balanced contiguous row blocks (pepp_partition_rows)."""
    rp = np.ascontiguousarray(row_ptr, dtype=np.int64)
    b = np.empty(nparts + 1, dtype=np.int64)
    C.check(C.lib().pepp_partition_rows(rp.ctypes.data, len(rp) - 1, int(rp[0]), nparts, b.ctypes.data),
            "pepp_partition_rows")
    return b


def halo_ghosts(col: np.ndarray, nranks: int, rank: int, row_bounds: Sequence[int]) -> tuple[np.ndarray, np.ndarray]:
    """(counts per owner rank, sorted ghost columns) of one row block."""
    c = np.ascontiguousarray(col, dtype=np.int32)
    rb = np.ascontiguousarray(row_bounds, dtype=np.int64)
    counts = np.zeros(nranks, dtype=np.int64)
    total = ctypes.c_int64()
    C.check(C.lib().pepp_halo_ghosts(c.ctypes.data if c.size else None, c.size, nranks, rank, rb.ctypes.data,
                                     counts.ctypes.data, None, 0, ctypes.byref(total)), "pepp_halo_ghosts")
    g = np.empty(max(1, total.value), dtype=np.int32)
    C.check(C.lib().pepp_halo_ghosts(c.ctypes.data if c.size else None, c.size, nranks, rank, rb.ctypes.data,
                                     counts.ctypes.data, g.ctypes.data, g.size, ctypes.byref(total)),
            "pepp_halo_ghosts")
    return counts, g[:total.value]


def dist_choose(means, eligible=None) -> tuple[int, np.ndarray]:
    """pepp_dist_choose: means [nranks][nd] (each rank's own mean µs per
    distribution candidate) -> (argmin of the max-over-ranks means, agreed)."""
    m = np.ascontiguousarray(means, dtype=np.float64)
    if m.ndim != 2:
        raise ValueError("means must be [nranks][nd]")
    e = None if eligible is None else np.ascontiguousarray([1 if v else 0 for v in eligible], dtype=np.uint8)
    ag = np.zeros(m.shape[1])
    c = ctypes.c_int32()
    C.check(C.lib().pepp_dist_choose(m.shape[0], m.shape[1], m.ctypes.data, e.ctypes.data if e is not None else None,
                                     ctypes.byref(c), ag.ctypes.data), "pepp_dist_choose")
    return c.value, ag


def context_key(nrows: int, ncols: int, nnz: int, cv: float, nparts: int = 1, *, f32: bool = False,
                compress: bool = False) -> int:
    inst = (C.KEY_F32 if f32 else 0) | (C.KEY_COMPRESS if compress else 0)
    return int(C.lib().pepp_context_key(nrows, ncols, nnz, cv, nparts, inst))


def nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    C.check(C.lib().pepp_nccl_unique_id(ctypes.addressof(buf)), "pepp_nccl_unique_id")
    return buf.raw


def nccl_selftest(device: int = -1) -> None:
    """Run every NCCL call of the partitioned path on a one-rank communicator
    and check the data (pepp_nccl_selftest); raises PeppError on mismatch."""
    C.check(C.lib().pepp_nccl_selftest(device), "pepp_nccl_selftest")
