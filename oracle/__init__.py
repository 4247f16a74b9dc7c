"""CPU oracle for the gSWORD hot path — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package.  The product package
(paper_journals_pacmmod_yelsg24_b200) never imports it and shares no code with it.

* oracle.c      — plain C sampler (WanderJoin P:L538, Alley P:L540, HT Eq. 1
                  P:L754) with its own Philox4x32-10, plus an exact backtracking
                  embedding counter.  Built into liboracle.so by `build()`.
* this module   — ctypes marshalling, multi-threaded sample ranges (the CPU
                  baselines' dynamic scheduling) and the aggregation of
                  Eq. 1 with a correctly rounded sum (math.fsum).
* exact.py      — pure-Python brute force and the exact enumeration-tree walk.

Parity status per function: see DESIGN.md §4 (all pinned; none "parity unpinned").
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
import threading
from concurrent.futures import ThreadPoolExecutor
from typing import Dict, Optional, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")
_lock = threading.Lock()
_lib = None

WJ = 0
ALLEY = 1
MAX_QV = 16

# per-sample record: restated from the layout contract (152 bytes)
RECORD_DTYPE = np.dtype([
    ("sample_id", "<u8"), ("valid", "u1"), ("depth_reached", "u1"), ("pad", "u1", (2,)),
    ("sectors", "<u4"),
    ("path", "<i4", (MAX_QV,)), ("csize", "<u4", (MAX_QV,)), ("weight", "<f8"),
])
assert RECORD_DTYPE.itemsize == 152

# trawling record (168 bytes): status 0 prefix died, 1 enumerated, 2 budget exceeded
TRAWL_DTYPE = np.dtype([
    ("sample_id", "<u8"), ("status", "u1"), ("d", "u1"), ("pad", "u1", (6,)),
    ("path", "<i4", (MAX_QV,)), ("csize", "<u4", (MAX_QV,)), ("weight", "<f8"), ("count", "<u8"),
    ("nodes", "<u8"),
])
assert TRAWL_DTYPE.itemsize == 168


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so (gcc, plain -O2)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-Wextra", "-shared", "-fPIC", "-pthread",
                               "-o", _SO, _SRC])
    return _SO


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_SO)
            P = ctypes.c_void_p
            lib.or_philox4x32_10.argtypes = [P, P, P]
            lib.or_philox4x32_10.restype = None
            lib.or_uniform_index.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint64]
            lib.or_uniform_index.restype = ctypes.c_uint64
            lib.or_sample_range.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_int32, P, P, P, P,
                                            ctypes.c_int, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64,
                                            P, P]
            lib.or_sample_range.restype = ctypes.c_int
            lib.or_sample_range_f.argtypes = lib.or_sample_range.argtypes + [ctypes.c_int]
            lib.or_sample_range_f.restype = ctypes.c_int
            lib.or_sample_range_v.argtypes = lib.or_sample_range_f.argtypes + [ctypes.c_int]
            lib.or_sample_range_v.restype = ctypes.c_int
            lib.or_sample_range_mt.argtypes = lib.or_sample_range_v.argtypes + [ctypes.c_int, ctypes.c_uint64]
            lib.or_sample_range_mt.restype = ctypes.c_int
            lib.or_candidate_sets.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_int32, P, P, P, P, ctypes.c_int, P]
            lib.or_candidate_sets.restype = ctypes.c_int
            lib.or_trawl_range.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_int32, P, P, P, P, ctypes.c_int,
                                           ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64,
                                           ctypes.c_int, P, P, P]
            lib.or_trawl_range.restype = ctypes.c_int
            lib.or_trawl_record_size.restype = ctypes.c_int
            assert lib.or_trawl_record_size() == TRAWL_DTYPE.itemsize
            lib.or_inherit_range.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_int32, P, P, P, P, ctypes.c_int,
                                             ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int, P, P]
            lib.or_inherit_range.restype = ctypes.c_int
            lib.or_inherit_range_v.argtypes = lib.or_inherit_range.argtypes + [ctypes.c_int]
            lib.or_inherit_range_v.restype = ctypes.c_int
            lib.or_count_embeddings.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_int32, P, P, P, P, P, P]
            lib.or_count_embeddings.restype = ctypes.c_int
            lib.or_record_size.restype = ctypes.c_int
            assert lib.or_record_size() == RECORD_DTYPE.itemsize
            _lib = lib
    return _lib


def _ptr(a: np.ndarray) -> ctypes.c_void_p:
    return ctypes.c_void_p(a.ctypes.data)


def philox4x32_10(ctr, key) -> Tuple[int, int, int, int]:
    lib = _load()
    c = np.asarray(ctr, np.uint32)
    k = np.asarray(key, np.uint32)
    o = np.zeros(4, np.uint32)
    lib.or_philox4x32_10(_ptr(c), _ptr(k), _ptr(o))
    return tuple(int(x) for x in o)


def uniform_index(seed: int, sid: int, d: int, c: int) -> int:
    return int(_load().or_uniform_index(seed, sid, d, c))


class _Prepared:
    """Contiguous typed copies of a graph and a query for the C calls."""

    def __init__(self, g, q):
        self.n = int(g.row_ptr.shape[0] - 1)
        self.row_ptr = np.ascontiguousarray(g.row_ptr, np.int64)
        self.col = np.ascontiguousarray(g.col, np.int32)
        self.labels = np.ascontiguousarray(g.labels, np.int32)
        qrp, qcol = q.csr()
        self.nq = int(q.nq)
        self.qrp = np.ascontiguousarray(qrp, np.int32)
        self.qcol = np.ascontiguousarray(qcol if qcol.shape[0] else np.zeros(1, np.int32), np.int32)
        self.qlab = np.ascontiguousarray(q.labels, np.int32)
        self.order = np.ascontiguousarray(q.order, np.int32)


FILTER_LABEL = 0
FILTER_LDF = 1
FILTER_NLF = 2

# Alley selection rule: count-then-index (default) or warp streaming (Alg. 3, reading A25)
SELECT_INDEX = 0
SELECT_STREAM = 1
# comparison variants of readings A3 / A5 (bit flags, combined with the selection rule)
VARIANT_WJ_PARENT_FIRST = 2
VARIANT_ALLEY_DUPCHECK_POST = 4


def candidate_sets(g, q, filter: int) -> np.ndarray:
    """C(u) membership, bool[nq, n] (Def. 4; filter per reading A21)."""
    lib = _load()
    pr = _Prepared(g, q)
    out = np.zeros((pr.nq, pr.n), np.uint8)
    rc = lib.or_candidate_sets(pr.n, _ptr(pr.row_ptr), _ptr(pr.col), _ptr(pr.labels), pr.nq, _ptr(pr.qrp),
                               _ptr(pr.qcol), _ptr(pr.qlab), _ptr(pr.order), int(filter), _ptr(out))
    if rc != 0:
        raise ValueError(f"oracle rejected input (rc={rc})")
    return out.astype(bool)


def sample_range(g, q, method: int, seed: int, first: int, count: int, records: bool = True,
                 threads: int = 1, filter: int = FILTER_LABEL, select: int = SELECT_INDEX,
                 variant: int = 0) -> Tuple[np.ndarray, Optional[np.ndarray]]:
    """Y values (and records) of samples [first, first+count), in sample-id order.
    select: Alley's selection rule, SELECT_INDEX (count-then-index) or SELECT_STREAM (warp
    streaming, Alg. 3, reading A25).  variant: VARIANT_* bits (readings A3, A5)."""
    lib = _load()
    pr = _Prepared(g, q)
    y = np.zeros(count, np.float64)
    rec = np.zeros(count, RECORD_DTYPE) if records else None

    # dynamic scheduling over chunks of sample ids on `threads` host threads; the
    # candidate sets are built once per call and shared by the threads
    threads = max(1, int(threads))
    chunk = max(1, min(1024, -(-count // (4 * threads)))) if threads > 1 else max(1, count)
    rc = lib.or_sample_range_mt(pr.n, _ptr(pr.row_ptr), _ptr(pr.col), _ptr(pr.labels), pr.nq, _ptr(pr.qrp),
                                _ptr(pr.qcol), _ptr(pr.qlab), _ptr(pr.order), int(method), int(seed), int(first),
                                int(count), _ptr(y), _ptr(rec) if records else None, int(filter),
                                int(select) | int(variant), threads, chunk) if count else 0
    if rc != 0:
        raise ValueError(f"oracle rejected input (rc={rc})")
    return y, rec


def trawl_range(g, q, method: int, seed: int, first: int, count: int, budget: int = 2**62, filter: int = 0,
                records: bool = True, threads: int = 1):
    """Trawling (Alg. 4; reading A23): T values, statuses, records."""
    lib = _load()
    pr = _Prepared(g, q)
    t = np.zeros(count, np.float64)
    st = np.zeros(count, np.uint8)
    rec = np.zeros(count, TRAWL_DTYPE) if records else None

    def run(a: int, b: int) -> int:
        return lib.or_trawl_range(pr.n, _ptr(pr.row_ptr), _ptr(pr.col), _ptr(pr.labels), pr.nq, _ptr(pr.qrp),
                                  _ptr(pr.qcol), _ptr(pr.qlab), _ptr(pr.order), int(method), int(seed),
                                  int(first + a), int(b - a), int(budget), int(filter),
                                  ctypes.c_void_p(t.ctypes.data + 8 * a), ctypes.c_void_p(st.ctypes.data + a),
                                  ctypes.c_void_p(rec.ctypes.data + TRAWL_DTYPE.itemsize * a) if records else None)

    if threads <= 1 or count < 2 * threads:
        rc = run(0, count) if count else 0
    else:
        chunk = max(1, min(65536, count // (threads * 8) or 1))
        bounds = [(a, min(count, a + chunk)) for a in range(0, count, chunk)]
        with ThreadPoolExecutor(max_workers=threads) as ex:
            rcs = list(ex.map(lambda ab: run(*ab), bounds))
        rc = min(rcs) if rcs else 0
    if rc != 0:
        raise ValueError(f"oracle rejected input (rc={rc})")
    return t, st, rec


def inherit_range(g, q, method: int, seed: int, first: int, count: int, filter: int = 0,
                  select: int = 0, variant: int = 0) -> Dict[str, float]:
    """Sample inheritance (Alg. 2) over groups of 32 consecutive ids (reading A24).
    estimate = sum of group totals / count; variance from the group totals (the groups are
    the independent units): m (sum G^2 - (sum G)^2 / m) / ((m - 1) count^2)."""
    lib = _load()
    pr = _Prepared(g, q)
    m = (count + 31) // 32
    groups = np.zeros(max(m, 1), np.float64)
    nc = np.zeros(1, np.uint64)
    rc = lib.or_inherit_range_v(pr.n, _ptr(pr.row_ptr), _ptr(pr.col), _ptr(pr.labels), pr.nq, _ptr(pr.qrp),
                                _ptr(pr.qcol), _ptr(pr.qlab), _ptr(pr.order), int(method), int(seed), int(first),
                                int(count), int(filter), _ptr(groups), _ptr(nc), int(select) | int(variant))
    if rc != 0:
        raise ValueError(f"oracle rejected input (rc={rc})")
    groups = groups[:m]
    s = math.fsum(groups.tolist())
    sq = math.fsum((groups * groups).tolist())
    var = m * (sq - s * s / m) / ((m - 1) * count * count) if m >= 2 else float("nan")
    return {"sum": s, "sumsq": sq, "n": count, "groups": m, "n_valid": int(nc[0]), "estimate": s / count,
            "variance": var, "group_totals": groups}


def trawl_aggregate(t: np.ndarray, status: np.ndarray) -> Dict[str, float]:
    """Trawling estimate: mean of T over the samples whose enumeration finished (the
    paper keeps only completed enumerations); timeouts reported separately."""
    done = status != 2
    agg = aggregate(t[done])
    agg["n_timeout"] = int(np.count_nonzero(~done))
    return agg


def aggregate(y: np.ndarray) -> Dict[str, float]:
    """HT estimator of Eq. 1: H = (1/n) sum_i Y_i; dead samples count in n
    (reading A8, Ex. 2 P:L758).  Sums are correctly rounded (math.fsum).  Variance of
    the estimator (reading A9): (sumsq - sum^2/n) / (n (n-1))."""
    y = np.asarray(y, np.float64)
    n = int(y.shape[0])
    s = math.fsum(y.tolist())
    sq = math.fsum((y * y).tolist())
    valid = int(np.count_nonzero(y))
    est = s / n if n else float("nan")
    var = (sq - s * s / n) / (n * (n - 1)) if n >= 2 else float("nan")
    return {"sum": s, "sumsq": sq, "n": n, "n_valid": valid, "estimate": est, "variance": var}


def estimate(g, q, method: int, seed: int, n_samples: int, first: int = 0, threads: int = 1,
             filter: int = FILTER_LABEL, select: int = 0, variant: int = 0) -> Dict[str, float]:
    y, _ = sample_range(g, q, method, seed, first, n_samples, records=False, threads=threads, filter=filter,
                        select=select, variant=variant)
    return aggregate(y)


def count_embeddings(g, q) -> int:
    """Exact number of (non-induced, labelled) embeddings of q in G (reading A1)."""
    lib = _load()
    pr = _Prepared(g, q)
    lo = np.zeros(1, np.uint64)
    hi = np.zeros(1, np.uint64)
    rc = lib.or_count_embeddings(pr.n, _ptr(pr.row_ptr), _ptr(pr.col), _ptr(pr.labels), pr.nq,
                                 _ptr(pr.qrp), _ptr(pr.qcol), _ptr(pr.qlab), _ptr(pr.order),
                                 _ptr(lo), _ptr(hi))
    if rc != 0:
        raise ValueError(f"oracle rejected input (rc={rc})")
    return (int(hi[0]) << 64) | int(lo[0])


def qerror(c: float, c_hat: float) -> float:
    """q-error: max(max(1,c)/max(1,c^), max(1,c^)/max(1,c))."""
    a = max(1.0, float(c))
    b = max(1.0, float(c_hat))
    return max(a / b, b / a)
