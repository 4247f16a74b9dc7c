"""ctypes binding of the gSWORD C ABI (include/gsword.h) — argument marshalling only.

Every step of the hot path runs in libgsword.so (sm_100a kernels + C++ host).  If
the library is missing this module raises at import: there is no CPU fallback.
Names follow the C ABI one to one: gsword_load_graph -> Context.load_graph, etc.
"""
from __future__ import annotations

import ctypes
import os
from typing import Dict, Optional, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# GSWORD_LIB overrides the library path (build-variant experiments only)
LIB_PATH = os.environ.get("GSWORD_LIB") or os.path.join(_HERE, "libgsword.so")

WJ = 0
ALLEY = 1
METHODS = {"wj": WJ, "wanderjoin": WJ, "alley": ALLEY, "al": ALLEY}
MAX_QV = 16

OPT_BLOCKS_PER_SM = 0
OPT_THREADS = 1
OPT_CHUNK = 2
OPT_L2_PERSIST = 3
OPT_COOP_THRESHOLD = 4
OPT_BLOOM = 5
OPT_EDGE_SET = 6
OPT_FILTER = 7
OPT_SCHEDULE = 8
OPT_REFILL_MIN = 9
OPT_AUTOTUNE = 10
OPT_BLOOM_BITS = 11
OPT_STREAMING = 12  # Alley by warp streaming (Alg. 3, reading A25)
OPT_VARIANT = 13  # comparison variants of readings A3/A5 (bit flags below)
OPT_OCCUPANCY = 14  # estimate-kernel occupancy variant: -1 autotuned, 0/1/2 forced
OPT_FAULT_QUEUE = 15  # fault injection: the next launch's queue starts here (one-shot)
OPT_TRAWL_WARP = 16  # trawl_range: 1 warp-cooperative enumeration (default), 0 one lane per sample
VARIANT_WJ_PARENT_FIRST = 2
VARIANT_ALLEY_DUPCHECK_POST = 4
SCHED_REFILL, SCHED_SAMPLE_SYNC, SCHED_INHERIT = 0, 1, 2
FILTER_LABEL, FILTER_LDF, FILTER_NLF = 0, 1, 2
CUDA_STREAM_LEGACY = 0x1  # cudaStreamLegacy

STATUS = {0: "OK", -1: "EINVAL", -2: "ENOGRAPH", -3: "ENOQUERY", -4: "EORDER", -5: "EGRAPH",
          -6: "ELIMIT", -7: "ECUDA", -8: "ENOMEM", -9: "EFAULT"}

# gsword_sample_record (152 bytes)
RECORD_DTYPE = np.dtype([
    ("sample_id", "<u8"), ("valid", "u1"), ("depth_reached", "u1"), ("pad", "u1", (2,)),
    ("sectors", "<u4"),
    ("path", "<i4", (MAX_QV,)), ("csize", "<u4", (MAX_QV,)), ("weight", "<f8"),
])
assert RECORD_DTYPE.itemsize == 152

# gsword_trawl_record (168 bytes)
TRAWL_DTYPE = np.dtype([
    ("sample_id", "<u8"), ("status", "u1"), ("d", "u1"), ("pad", "u1", (6,)),
    ("path", "<i4", (MAX_QV,)), ("csize", "<u4", (MAX_QV,)), ("weight", "<f8"), ("count", "<u8"),
    ("nodes", "<u8"),
])
assert TRAWL_DTYPE.itemsize == 168


class GswordError(RuntimeError):
    def __init__(self, status: int, message: str):
        super().__init__(f"gsword {STATUS.get(status, status)}: {message}")
        self.status = status


class _Result(ctypes.Structure):
    _fields_ = [("estimate", ctypes.c_double), ("variance", ctypes.c_double), ("sum", ctypes.c_double),
                ("sumsq", ctypes.c_double), ("n_samples", ctypes.c_uint64), ("n_valid", ctypes.c_uint64),
                ("seconds", ctypes.c_double)]


class _QueryStats(ctypes.Structure):
    _fields_ = [("nq", ctypes.c_int32), ("filter", ctypes.c_int32), ("candidates", ctypes.c_uint64 * MAX_QV),
                ("cg_entries", ctypes.c_uint64), ("build_seconds", ctypes.c_double),
                ("refill_min", ctypes.c_int32 * 2), ("occupancy", ctypes.c_int32 * 2), ("cg_bytes", ctypes.c_uint64)]


class _PlanInfo(ctypes.Structure):
    _fields_ = [("nq", ctypes.c_int32), ("label", ctypes.c_int32 * MAX_QV),
                ("back_mask", ctypes.c_uint32 * MAX_QV), ("dup_mask", ctypes.c_uint32 * MAX_QV)]


def _load_library() -> ctypes.CDLL:
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `make` (or __graft_entry__.build()); "
                          "there is no CPU fallback for the gSWORD hot path")
    lib = ctypes.CDLL(LIB_PATH)
    P = ctypes.c_void_p
    I32, I64, U64 = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64
    sig = {
        "gsword_create": ([ctypes.c_int, ctypes.POINTER(P)], ctypes.c_int),
        "gsword_destroy": ([P], ctypes.c_int),
        "gsword_set_stream": ([P, P], ctypes.c_int),
        "gsword_set_option": ([P, ctypes.c_int, I64], ctypes.c_int),
        "gsword_load_graph": ([P, I64, P, P, P, I32], ctypes.c_int),
        "gsword_load_query": ([P, I32, P, P, P, P], ctypes.c_int),
        "gsword_load_graph_device": ([P, I64, P, P, P, I32], ctypes.c_int),
        "gsword_estimate": ([P, ctypes.c_int, U64, U64, ctypes.POINTER(_Result)], ctypes.c_int),
        "gsword_estimate_range": ([P, ctypes.c_int, U64, U64, U64, ctypes.POINTER(_Result)], ctypes.c_int),
        "gsword_estimate_async": ([P, ctypes.c_int, U64, U64, U64, P], ctypes.c_int),
        "gsword_estimate_until": ([P, ctypes.c_int, U64, ctypes.c_double, U64, U64, ctypes.POINTER(_Result)],
                                  ctypes.c_int),
        "gsword_finalize": ([P, ctypes.POINTER(_Result)], ctypes.c_int),
        "gsword_trace_samples": ([P, ctypes.c_int, U64, U64, U64, P], ctypes.c_int),
        "gsword_count_sectors": ([P, ctypes.c_int, U64, U64, U64, P, P], ctypes.c_int),
        "gsword_launch_info": ([P, P, P, P], ctypes.c_int),
        "gsword_gather_roofline": ([P, U64, ctypes.c_int, P], ctypes.c_int),
        "gsword_last_kernel_seconds": ([P, P], ctypes.c_int),
        "gsword_phase_cycles": ([P, P], ctypes.c_int),
        "gsword_query_info": ([P, ctypes.POINTER(_QueryStats)], ctypes.c_int),
        "gsword_quicksi_order": ([I64, P, P, P, I32, I32, P, P, P, P], ctypes.c_int),
        "gsword_trawl_range": ([P, ctypes.c_int, U64, U64, U64, U64, ctypes.POINTER(_Result), P], ctypes.c_int),
        "gsword_trace_trawl": ([P, ctypes.c_int, U64, U64, U64, U64, P], ctypes.c_int),
        "gsword_select_order": ([P, ctypes.c_int, ctypes.c_int, I32, P, P, P, U64, U64, P, P], ctypes.c_int),
        "gsword_check_graph": ([I64, P, P, P, I32], ctypes.c_int),
        "gsword_plan_query": ([I32, P, P, P, P, I32, ctypes.POINTER(_PlanInfo)], ctypes.c_int),
        "gsword_last_error": ([], ctypes.c_char_p),
        "gsword_version": ([], ctypes.c_int),
    }
    for name, (args, res) in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    return lib


_lib = _load_library()


def _check(rc: int) -> None:
    if rc != 0:
        raise GswordError(rc, _lib.gsword_last_error().decode())


def _ptr(a: Optional[np.ndarray]):
    return None if a is None else ctypes.c_void_p(a.ctypes.data)


def version() -> int:
    return int(_lib.gsword_version())


def _result_dict(r: _Result) -> Dict[str, float]:
    return {"estimate": r.estimate, "variance": r.variance, "sum": r.sum, "sumsq": r.sumsq,
            "n": int(r.n_samples), "n_valid": int(r.n_valid), "seconds": r.seconds}


def finalize(values4) -> Dict[str, float]:
    """gsword_finalize: {sum, sumsq, n_valid, n} -> estimate / variance (Eq. 1)."""
    h = np.ascontiguousarray(np.asarray(values4, dtype=np.float64).reshape(4))
    r = _Result()
    _check(_lib.gsword_finalize(_ptr(h), ctypes.byref(r)))
    return _result_dict(r)


def check_graph(row_ptr, col, labels=None, n_labels: int = 1) -> None:
    rp = np.ascontiguousarray(row_ptr, np.int64)
    cl = np.ascontiguousarray(col, np.int32)
    lb = None if labels is None else np.ascontiguousarray(labels, np.int32)
    _check(_lib.gsword_check_graph(rp.shape[0] - 1, _ptr(rp), _ptr(cl), _ptr(lb), int(n_labels)))


def _query_arrays(q_row_ptr, q_col, q_labels, order):
    qrp = np.ascontiguousarray(q_row_ptr, np.int32)
    qcol = np.ascontiguousarray(q_col, np.int32)
    if qcol.shape[0] == 0:
        qcol = np.zeros(1, np.int32)
    qlab = np.ascontiguousarray(q_labels, np.int32)
    od = np.ascontiguousarray(order, np.int32)
    return qrp, qcol, qlab, od


def plan_query(q_row_ptr, q_col, q_labels, order, n_labels: int) -> Dict[str, list]:
    qrp, qcol, qlab, od = _query_arrays(q_row_ptr, q_col, q_labels, order)
    info = _PlanInfo()
    _check(_lib.gsword_plan_query(qlab.shape[0], _ptr(qrp), _ptr(qcol), _ptr(qlab), _ptr(od), int(n_labels),
                                  ctypes.byref(info)))
    nq = info.nq
    return {"nq": nq, "label": list(info.label)[:nq], "back_mask": list(info.back_mask)[:nq],
            "dup_mask": list(info.dup_mask)[:nq]}


ORDER_QUICKSI = 0
ORDER_TRIAL = 1


def quicksi_order(row_ptr, col, labels, n_labels, q_row_ptr, q_col, q_labels) -> list:
    """gsword_quicksi_order: infrequent-edge-first matching order (host only, reading A22)."""
    rp = np.ascontiguousarray(row_ptr, np.int64)
    cl = np.ascontiguousarray(col, np.int32)
    if cl.shape[0] == 0:
        cl = np.zeros(1, np.int32)
    lb = None if labels is None or n_labels == 1 else np.ascontiguousarray(labels, np.int32)
    qrp, qcol, qlab, _ = _query_arrays(q_row_ptr, q_col, q_labels, np.zeros(1, np.int32))
    out = np.zeros(qlab.shape[0], np.int32)
    _check(_lib.gsword_quicksi_order(rp.shape[0] - 1, _ptr(rp), _ptr(cl), _ptr(lb), int(n_labels), qlab.shape[0],
                                     _ptr(qrp), _ptr(qcol), _ptr(qlab), _ptr(out)))
    return out.tolist()


def qerror(c: float, c_hat: float) -> float:
    """q-error: max(max(1,c)/max(1,c^), max(1,c^)/max(1,c))."""
    a = max(1.0, float(c))
    b = max(1.0, float(c_hat))
    return max(a / b, b / a)


class Context:
    """One gsword_ctx on one CUDA device.  Methods mirror the C ABI."""

    def __init__(self, device: int = 0):
        h = ctypes.c_void_p()
        _check(_lib.gsword_create(int(device), ctypes.byref(h)))
        self._h = h
        self.device = device
        self.nq = 0

    def close(self) -> None:
        if getattr(self, "_h", None):
            _lib.gsword_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    # -- configuration --------------------------------------------------------------
    def set_stream(self, stream) -> None:
        """stream: torch.cuda.Stream, an int cudaStream_t, or None for the context's own.
        A handle of 0 (torch's default stream) maps to cudaStreamLegacy."""
        if stream is None:
            _check(_lib.gsword_set_stream(self._h, None))
            return
        handle = int(getattr(stream, "cuda_stream", stream))
        _check(_lib.gsword_set_stream(self._h, ctypes.c_void_p(handle if handle else CUDA_STREAM_LEGACY)))

    def set_option(self, option: int, value: int) -> None:
        _check(_lib.gsword_set_option(self._h, int(option), int(value)))

    def gather_roofline(self, buffer_bytes: int, inflight: int = 8) -> float:
        """Sustained random 32-byte-sector gather rate (sectors/s) over a buffer of that size."""
        out = ctypes.c_double()
        _check(_lib.gsword_gather_roofline(self._h, int(buffer_bytes), int(inflight), ctypes.byref(out)))
        return out.value

    def launch_info(self) -> Dict[str, int]:
        g, t, l = ctypes.c_int(), ctypes.c_int(), ctypes.c_int()
        _check(_lib.gsword_launch_info(self._h, ctypes.byref(g), ctypes.byref(t), ctypes.byref(l)))
        return {"grid": g.value, "threads": t.value, "launches_per_estimate": l.value}

    def phase_cycles(self) -> list:
        out = (ctypes.c_double * 8)()
        _check(_lib.gsword_phase_cycles(self._h, out))
        return list(out)

    def last_kernel_seconds(self) -> float:
        out = ctypes.c_double()
        _check(_lib.gsword_last_kernel_seconds(self._h, ctypes.byref(out)))
        return out.value

    # -- graph / query ----------------------------------------------------------------
    def load_graph(self, row_ptr, col, labels=None, n_labels: int = 1) -> None:
        rp = np.ascontiguousarray(row_ptr, np.int64)
        cl = np.ascontiguousarray(col, np.int32)
        if cl.shape[0] == 0:
            cl = np.zeros(1, np.int32)
        lb = None if labels is None or n_labels == 1 else np.ascontiguousarray(labels, np.int32)
        _check(_lib.gsword_load_graph(self._h, rp.shape[0] - 1, _ptr(rp), _ptr(cl), _ptr(lb), int(n_labels)))

    def load_graph_device(self, row_ptr, col, labels=None, n_labels: int = 1) -> None:
        """gsword_load_graph_device: CUDA tensors (int64 row_ptr, int32 col label-sorted per
        row, int32 labels or None) on this context's device; col/labels are borrowed and kept
        referenced here until the next load."""
        for t in (row_ptr, col) + ((labels,) if labels is not None else ()):
            if not t.is_cuda or not t.is_contiguous():
                raise ValueError("load_graph_device needs contiguous CUDA tensors")
        lab_ptr = ctypes.c_void_p(labels.data_ptr()) if labels is not None and n_labels > 1 else None
        _check(_lib.gsword_load_graph_device(self._h, int(row_ptr.numel() - 1), ctypes.c_void_p(row_ptr.data_ptr()),
                                             ctypes.c_void_p(col.data_ptr()), lab_ptr, int(n_labels)))
        self._borrowed = (col, labels)

    def load_query(self, q_row_ptr, q_col, q_labels, order) -> int:
        """Returns the bytes handed to the library (query CSR + labels + order)."""
        qrp, qcol, qlab, od = _query_arrays(q_row_ptr, q_col, q_labels, order)
        _check(_lib.gsword_load_query(self._h, qlab.shape[0], _ptr(qrp), _ptr(qcol), _ptr(qlab), _ptr(od)))
        self.nq = int(qlab.shape[0])
        return int(qrp.nbytes + qcol.nbytes + qlab.nbytes + od.nbytes)

    def select_order(self, strategy: int, method: int, q_row_ptr, q_col, q_labels, pilot_samples: int = 100_000,
                     seed: int = 1):
        """gsword_select_order: choose and LOAD a matching order; returns (order, score)."""
        qrp, qcol, qlab, _ = _query_arrays(q_row_ptr, q_col, q_labels, np.zeros(1, np.int32))
        out = np.zeros(qlab.shape[0], np.int32)
        score = ctypes.c_double()
        _check(_lib.gsword_select_order(self._h, int(strategy), int(method), qlab.shape[0], _ptr(qrp), _ptr(qcol),
                                        _ptr(qlab), int(pilot_samples), int(seed), _ptr(out), ctypes.byref(score)))
        self.nq = int(qlab.shape[0])
        return out.tolist(), score.value

    def query_info(self) -> Dict[str, object]:
        st = _QueryStats()
        _check(_lib.gsword_query_info(self._h, ctypes.byref(st)))
        return {"nq": st.nq, "filter": st.filter, "candidates": list(st.candidates)[:st.nq],
                "cg_entries": int(st.cg_entries), "build_seconds": st.build_seconds, "cg_bytes": int(st.cg_bytes),
                "refill_min": list(st.refill_min), "occupancy": list(st.occupancy)}

    # convenience for workloads.gen.Graph / Query objects
    def load_graph_obj(self, g) -> None:
        self.load_graph(g.row_ptr, g.col, g.labels, g.n_labels)

    def load_query_obj(self, q) -> int:
        qrp, qcol = q.csr()
        return self.load_query(qrp, qcol, q.labels, q.order)

    # -- estimation ---------------------------------------------------------------------
    def estimate(self, method: int, n_samples: int, seed: int, first: int = 0) -> Dict[str, float]:
        r = _Result()
        _check(_lib.gsword_estimate_range(self._h, int(method), int(first), int(n_samples), int(seed),
                                          ctypes.byref(r)))
        return _result_dict(r)

    def estimate_until(self, method: int, seed: int, rel_se: float, min_samples: int = 1_000_000,
                       max_samples: int = 10**10) -> Dict[str, float]:
        """gsword_estimate_until: sample until the relative standard error reaches rel_se."""
        r = _Result()
        _check(_lib.gsword_estimate_until(self._h, int(method), int(seed), float(rel_se), int(min_samples),
                                          int(max_samples), ctypes.byref(r)))
        return _result_dict(r)

    def estimate_async(self, method: int, first: int, n_samples: int, seed: int, out4) -> None:
        """Enqueue; out4 is a device pointer (int) or a CUDA tensor of 4 float64."""
        ptr = out4.data_ptr() if hasattr(out4, "data_ptr") else int(out4)
        _check(_lib.gsword_estimate_async(self._h, int(method), int(first), int(n_samples), int(seed),
                                          ctypes.c_void_p(ptr)))

    def trawl(self, method: int, n_samples: int, seed: int, first: int = 0, node_budget: int = 2**62):
        """gsword_trawl_range: trawling estimate (Alg. 4) over [first, first+n)."""
        r = _Result()
        to = ctypes.c_uint64()
        _check(_lib.gsword_trawl_range(self._h, int(method), int(first), int(n_samples), int(seed),
                                       int(node_budget), ctypes.byref(r), ctypes.byref(to)))
        out = _result_dict(r)
        out["n_timeout"] = int(to.value)
        return out

    def trace_trawl(self, method: int, first: int, n_samples: int, seed: int, node_budget: int = 2**62):
        rec = np.zeros(int(n_samples), TRAWL_DTYPE)
        _check(_lib.gsword_trace_trawl(self._h, int(method), int(first), int(n_samples), int(seed),
                                       int(node_budget), _ptr(rec)))
        return rec

    def trace_samples(self, method: int, first: int, n_samples: int, seed: int) -> np.ndarray:
        rec = np.zeros(int(n_samples), RECORD_DTYPE)
        _check(_lib.gsword_trace_samples(self._h, int(method), int(first), int(n_samples), int(seed),
                                         _ptr(rec)))
        return rec

    def count_sectors(self, method: int, first: int, n_samples: int, seed: int) -> Tuple[float, float]:
        """(algorithmic sectors of reading A26, sectors this implementation touches) summed
        over samples [first, first + n_samples)."""
        out = ctypes.c_double()
        touched = ctypes.c_double()
        _check(_lib.gsword_count_sectors(self._h, int(method), int(first), int(n_samples), int(seed),
                                         ctypes.byref(out), ctypes.byref(touched)))
        return out.value, touched.value
