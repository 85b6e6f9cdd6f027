"""ctypes wrapper of the CPU oracle (oracle/liboracle.so).  TEST INFRASTRUCTURE ONLY.

Only tests/, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` / ``--impl reference``
legs may import this module.  The product path (paper_conf_ipps_jim11_b200) never does.
Semantics: SURVEY.md §8(c) C-1/C-2, PAPER.md L51-52 and L125 (see oracle.cpp header).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
WC, SM, KM, II, SML = 1, 2, 3, 4, 5
NAMES = {"wc": WC, "sm": SM, "km": KM, "ii": II, "sml": SML}   # sml: StringMatch per line (L125)


class _Result(C.Structure):
    _fields_ = [("n_keys", C.c_uint64), ("keys", C.c_void_p), ("key_offsets", C.c_void_p),
                ("vals", C.c_void_p), ("val_offsets", C.c_void_p)]


_LIB = None
_PATH = os.path.join(_HERE, "liboracle.so")   # the portable build (Makefile: -O3 -ffp-contract=off)
_FLAGS = "-O3 -ffp-contract=off (portable build)"


def use_native() -> str:
    """Switch to an oracle build for THIS host (-O3 -march=native
    -ffp-contract=off), compiled once into the temp directory; the arithmetic is the same source
    (no fast-math, no contraction).  Falls back to the portable build if g++ fails.  Returns the
    flags of the build in use."""
    global _PATH, _FLAGS, _LIB
    if _LIB is not None or "march=native" in _FLAGS:
        return _FLAGS
    import hashlib
    import subprocess
    import tempfile
    src = os.path.join(_HERE, "oracle.cpp")
    tag = hashlib.sha1(open(src, "rb").read() + os.uname().nodename.encode()).hexdigest()[:12]
    out = os.path.join(tempfile.gettempdir(), f"bmr_oracle_native_{tag}.so")
    flags = ["-O3", "-march=native", "-std=c++17", "-fPIC", "-shared", "-ffp-contract=off"]
    if not os.path.exists(out):
        r = subprocess.run(["g++", *flags, "-o", out + ".tmp", src], capture_output=True, text=True)
        if r.returncode != 0:
            return _FLAGS
        os.replace(out + ".tmp", out)
    _PATH, _FLAGS = out, " ".join(f for f in flags if f not in ("-fPIC", "-shared", "-std=c++17"))
    return _FLAGS


def build_flags() -> str:
    return _FLAGS


def lib():
    global _LIB
    if _LIB is None:
        path = _PATH
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run __graft_entry__.build()")
        L = C.CDLL(path)
        L.oracle_create.argtypes = [C.c_int, C.c_void_p, C.c_uint32, C.c_void_p]
        L.oracle_create.restype = C.c_void_p
        L.oracle_map.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_uint64, C.c_uint32, C.c_uint64]
        L.oracle_pairs.argtypes = [C.c_void_p]
        L.oracle_pairs.restype = C.c_uint64
        L.oracle_reduce.argtypes = [C.c_void_p, C.POINTER(_Result)]
        L.oracle_destroy.argtypes = [C.c_void_p]
        _LIB = L
    return _LIB


def _copy(ptr, n, dtype):
    if n == 0:
        return np.zeros(0, dtype)
    buf = (C.c_uint8 * (n * np.dtype(dtype).itemsize)).from_address(ptr)
    return np.frombuffer(buf, dtype=dtype).copy()


def run(workload, batches, pattern: bytes | None = None, centroids: np.ndarray | None = None) -> dict:
    """Run the oracle over ``batches`` = [(records u8, offsets u64 | None, n, stride, base), ...].

    Returns the canonical result {n_keys, keys, key_offsets, vals, val_offsets, pairs} with
    the mr_result encoding: WC key=word val=u64 count | SM key=u64 offset |
    KM key=u32 id val=8xf32 centroid + u64 count | II key=URL val=u64[] ascending.
    """
    L = lib()
    w = NAMES.get(workload, workload)
    pat = None
    if pattern is not None:
        pat = (C.c_uint8 * 16)(*pattern[:16])
    k = 0
    cen = None
    if centroids is not None:
        centroids = np.ascontiguousarray(centroids, np.float32)
        k = centroids.shape[0]
        cen = centroids.ctypes.data_as(C.c_void_p)
    job = L.oracle_create(w, pat, k, cen)
    if not job:
        raise ValueError("oracle_create failed")
    try:
        for rec, off, n, stride, base in batches:
            rec = np.ascontiguousarray(rec, np.uint8)
            offp = None
            if off is not None:
                off = np.ascontiguousarray(off, np.uint64)
                offp = off.ctypes.data_as(C.c_void_p)
            rc = L.oracle_map(job, rec.ctypes.data_as(C.c_void_p), offp, n, stride, base)
            if rc:
                raise ValueError(f"oracle_map rc={rc}")
        pairs = int(L.oracle_pairs(job))
        R = _Result()
        L.oracle_reduce(job, C.byref(R))
        nk = int(R.n_keys)
        ko = _copy(R.key_offsets, nk + 1, np.uint64)
        vo = _copy(R.val_offsets, nk + 1, np.uint64)
        return {"n_keys": nk, "keys": _copy(R.keys, int(ko[-1]), np.uint8), "key_offsets": ko,
                "vals": _copy(R.vals, int(vo[-1]), np.uint8), "val_offsets": vo, "pairs": pairs}
    finally:
        L.oracle_destroy(job)
