"""Seeded synthetic input generators (test / bench infrastructure, no MapReduce arithmetic).

Host side: ctypes over ``gen/libbmrgen.so`` (built from ``bmr_gen.h`` + ``gen_host.c``).
Device side: ``gen/libbmrgen_cuda.so`` (same header compiled for sm_100a), see ``device_*``.
Both produce identical bytes for the same spec / page range (tests/test_gen_device.py).

Config recipes follow SURVEY.md §8(d) D-1 and PAPER.md Table II (L195-270); seeds are
``0xB200BA5E ^ config_id``.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
SEED_BASE = 0xB200BA5E
PAGE = 1 << 20
SM_PATTERN = b"#needle:0123456#"
KM_DIM = 8


class TextParams(C.Structure):
    _fields_ = [
        ("seed", C.c_uint64), ("kind", C.c_uint32), ("page_bytes", C.c_uint32),
        ("line_base", C.c_uint32), ("line_u1", C.c_uint32), ("line_u2", C.c_uint32),
        ("vocab", C.c_uint32), ("punct_ppm", C.c_uint32), ("plant_ppm", C.c_uint32),
        ("pattern", C.c_uint8 * 16),
        ("zipf_q", C.c_void_p), ("zipf_qn", C.c_uint32),
        ("len_q", C.c_void_p), ("len_qn", C.c_uint32),
        ("url_q", C.c_void_p), ("url_qn", C.c_uint32),
        ("link_ppm", C.c_uint32), ("name_ppm", C.c_uint32), ("upper_ppm", C.c_uint32),
        ("unclosed_ppm", C.c_uint32),
    ]


TEXT, HTML = 1, 2
QN = 1 << 16


@dataclass
class TextSpec:
    """A text-like workload (WC / SM / II).  Records are '\\n'-terminated lines."""
    kind: int = TEXT
    seed: int = SEED_BASE ^ 1
    page_bytes: int = PAGE
    line_base: int = 27
    line_u1: int = 6
    line_u2: int = 7
    vocab: int = 10_000
    zipf_s: float = 1.0
    punct_ppm: int = 50_000
    plant_ppm: int = 0
    pattern: bytes = SM_PATTERN
    # II
    ln_mu: float = 3.382
    ln_sigma: float = 1.245
    ln_max: int = 65536
    url_space: int = 1 << 24
    url_s: float = 0.8
    link_ppm: int = int(round(1e6 / 7.94))
    name_ppm: int = 10_000
    upper_ppm: int = 10_000
    unclosed_ppm: int = 5_000
    _tables: dict = field(default_factory=dict, repr=False, compare=False)


def _lib():
    global _LIB
    try:
        return _LIB
    except NameError:
        pass
    path = os.path.join(_HERE, "libbmrgen.so")
    if not os.path.exists(path):
        raise RuntimeError(f"{path} missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = C.CDLL(path)
    L.bmrg_build_zipf_q.argtypes = [C.c_double, C.c_uint32, C.c_uint32, C.c_void_p]
    L.bmrg_build_lognormal_q.argtypes = [C.c_double, C.c_double, C.c_uint32, C.c_uint32, C.c_uint32, C.c_void_p]
    L.bmrg_km_centres.argtypes = [C.c_uint64, C.c_uint32, C.c_uint32, C.c_void_p]
    L.bmrg_host_pages.argtypes = [C.POINTER(TextParams), C.c_uint64, C.c_uint64, C.c_void_p, C.c_void_p,
                                  C.c_int, C.c_void_p, C.c_void_p, C.c_uint64, C.c_void_p,
                                  C.c_void_p, C.c_uint64, C.c_void_p]
    L.bmrg_host_offsets.argtypes = [C.c_void_p, C.c_uint64, C.c_uint32, C.c_void_p, C.c_void_p, C.c_int]
    L.bmrg_host_km.argtypes = [C.c_uint64, C.c_uint64, C.c_uint64, C.c_void_p, C.c_uint32, C.c_void_p, C.c_int]
    L.bmrg_host_word.argtypes = [C.c_uint32, C.c_void_p]
    L.bmrg_host_word.restype = C.c_uint32
    L.bmrg_host_url.argtypes = [C.c_uint32, C.c_void_p]
    L.bmrg_host_url.restype = C.c_uint32
    _LIB = L
    return L


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


def tables(spec: TextSpec) -> dict:
    """Quantile tables (host numpy u32 arrays), cached on the spec."""
    if spec._tables:
        return spec._tables
    L = _lib()
    t = {}
    if spec.kind == TEXT:
        q = np.zeros(QN + 1, np.uint32)
        L.bmrg_build_zipf_q(spec.zipf_s, spec.vocab, QN, _ptr(q))
        t["zipf_q"] = q
    else:
        q = np.zeros(QN + 1, np.uint32)
        L.bmrg_build_lognormal_q(spec.ln_mu, spec.ln_sigma, 1, spec.ln_max, QN, _ptr(q))
        t["len_q"] = q
        u = np.zeros(QN + 1, np.uint32)
        L.bmrg_build_zipf_q(spec.url_s, spec.url_space, QN, _ptr(u))
        t["url_q"] = u
    spec._tables = t
    return t


def params(spec: TextSpec, table_ptrs: dict | None = None) -> TextParams:
    """Fill the C struct.  ``table_ptrs`` overrides the table addresses (device copies)."""
    t = tables(spec)
    P = TextParams()
    P.seed = spec.seed & 0xFFFFFFFFFFFFFFFF
    P.kind = spec.kind
    P.page_bytes = spec.page_bytes
    P.line_base, P.line_u1, P.line_u2 = spec.line_base, spec.line_u1, spec.line_u2
    P.vocab = spec.vocab
    P.punct_ppm = spec.punct_ppm
    P.plant_ppm = spec.plant_ppm
    for i, b in enumerate(spec.pattern[:16].ljust(16, b"\0")):
        P.pattern[i] = b
    ptrs = table_ptrs or {k: int(v.ctypes.data) for k, v in t.items()}
    if spec.kind == TEXT:
        P.zipf_q, P.zipf_qn = ptrs["zipf_q"], QN
    else:
        P.len_q, P.len_qn = ptrs["len_q"], QN
        P.url_q, P.url_qn = ptrs["url_q"], QN
    P.link_ppm, P.name_ppm = spec.link_ppm, spec.name_ppm
    P.upper_ppm, P.unclosed_ppm = spec.upper_ppm, spec.unclosed_ppm
    return P


def _nthreads(n=None):
    if n:
        return n
    try:
        return max(1, len(os.sched_getaffinity(0)))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


def host_text(spec: TextSpec, npages: int, page0: int = 0, truth: bool = False,
              nthreads: int | None = None) -> dict:
    """Generate pages [page0, page0+npages): returns data (u8), offsets (u64, n+1, relative to
    the first byte of ``data``), n, base (global byte offset of data[0]) and optional truth."""
    L = _lib()
    P = params(spec)
    nb = npages * spec.page_bytes
    data = np.empty(nb, np.uint8)
    lines = np.zeros(npages, np.uint32)
    nt = _nthreads(nthreads)
    out = {"data": data, "base": page0 * spec.page_bytes}
    hist = np.zeros(spec.vocab, np.uint32) if (truth and spec.kind == TEXT) else None
    cap = max(1024, nb // 16) if truth else 0
    plants = np.zeros(cap, np.uint64) if (truth and spec.plant_ppm) else None
    links = np.zeros(cap, np.uint64) if (truth and spec.kind == HTML) else None
    npl = C.c_uint64(0)
    nli = C.c_uint64(0)
    rc = L.bmrg_host_pages(C.byref(P), page0, npages, _ptr(data), _ptr(lines), nt,
                           _ptr(hist) if hist is not None else None,
                           _ptr(plants) if plants is not None else None, cap, C.byref(npl),
                           _ptr(links) if links is not None else None, cap, C.byref(nli))
    if rc:
        raise RuntimeError(f"bmrg_host_pages rc={rc}")
    n = int(lines.sum())
    offsets = np.zeros(n + 1, np.uint64)
    L.bmrg_host_offsets(_ptr(data), npages, spec.page_bytes, _ptr(lines), _ptr(offsets), nt)
    out.update(offsets=offsets, n=n, page_lines=lines)
    if hist is not None:
        out["word_hist"] = hist
    if plants is not None:
        assert npl.value <= cap
        out["plants"] = np.sort(plants[: npl.value])
    if links is not None:
        assert nli.value <= cap
        out["links"] = np.sort(links[: nli.value])
    return out


def word(rank: int) -> bytes:
    buf = (C.c_uint8 * 16)()
    n = _lib().bmrg_host_word(rank, buf)
    return bytes(buf[:n])


def url(uid: int) -> bytes:
    buf = (C.c_uint8 * 520)()
    n = _lib().bmrg_host_url(uid, buf)
    return bytes(buf[:n])


# ---------------- KMeans ----------------
@dataclass
class KMSpec:
    seed: int = SEED_BASE ^ 3
    k: int = 32
    min_dist: int = 64
    init_offset: float = 0.5


def km_centres(spec: KMSpec) -> tuple[np.ndarray, np.ndarray]:
    """(blob centres int32 k x 8, initial centroids float32 k x 8 = centre + init_offset)."""
    c = np.zeros((spec.k, KM_DIM), np.int32)
    rc = _lib().bmrg_km_centres(spec.seed & 0xFFFFFFFFFFFFFFFF, spec.k, spec.min_dist, _ptr(c))
    if rc:
        raise RuntimeError(f"bmrg_km_centres rc={rc}")
    init = (c.astype(np.float32) + np.float32(spec.init_offset)).astype(np.float32)
    return c, init


def host_km(spec: KMSpec, n: int, i0: int = 0, nthreads: int | None = None) -> np.ndarray:
    c, _ = km_centres(spec)
    pts = np.empty((n, KM_DIM), np.float32)
    rc = _lib().bmrg_host_km(spec.seed & 0xFFFFFFFFFFFFFFFF, i0, n, _ptr(c), spec.k, _ptr(pts), _nthreads(nthreads))
    if rc:
        raise RuntimeError(f"bmrg_host_km rc={rc}")
    return pts


# ---------------- configs (BASELINE.json `configs`) ----------------
def spec_wc(vocab=10_000, cid=1) -> TextSpec:
    return TextSpec(kind=TEXT, seed=SEED_BASE ^ cid, vocab=vocab)


def spec_sm(plant_ppm=1000, cid=2) -> TextSpec:
    return TextSpec(kind=TEXT, seed=SEED_BASE ^ cid, line_base=39, line_u1=6, line_u2=7,
                    vocab=10_000, plant_ppm=plant_ppm)


def spec_ii(cid=4) -> TextSpec:
    return TextSpec(kind=HTML, seed=SEED_BASE ^ cid)


CONFIGS = {
    # name: (workload, spec factory, pages or points)
    "C1": ("wc", lambda: spec_wc(10_000, 1), 1),                 # 1 MiB WC, V=10k
    "C2": ("sm", lambda: spec_sm(1000, 2), 4096),                # 4 GiB SM
    "C3": ("km", lambda: KMSpec(seed=SEED_BASE ^ 3), 64 << 20),  # 64M points
    "C4": ("ii", lambda: spec_ii(4), 8192),                      # 8 GiB II
    "C5": ("wc", lambda: spec_wc(1_000_000, 5), 8192),           # 8 GiB per GPU, V=1M
}


# ---------------- device generation (torch tensors on cuda) ----------------
_CLIB = None


def _clib():
    global _CLIB
    if _CLIB is None:
        path = os.path.join(_HERE, "libbmrgen_cuda.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run __graft_entry__.build()")
        L = C.CDLL(path)
        L.bmrg_dev_pages.argtypes = [C.POINTER(TextParams), C.c_uint64, C.c_uint64, C.c_void_p, C.c_void_p, C.c_void_p]
        L.bmrg_dev_offsets.argtypes = [C.c_void_p, C.c_uint64, C.c_uint32, C.c_void_p, C.c_void_p, C.c_void_p]
        L.bmrg_dev_km.argtypes = [C.c_uint64, C.c_uint64, C.c_uint64, C.c_void_p, C.c_uint32, C.c_void_p, C.c_void_p]
        _CLIB = L
    return _CLIB


def device_text(spec: TextSpec, npages: int, page0: int = 0, device: str = "cuda") -> dict:
    """Same bytes as host_text, generated in HBM.  offsets is an int64 tensor holding the u64
    offsets (n+1 entries)."""
    import torch
    L = _clib()
    t = tables(spec)
    dt = {k: torch.from_numpy(v.astype(np.uint32).view(np.int32)).to(device) for k, v in t.items()}
    P = params(spec, {k: v.data_ptr() for k, v in dt.items()})
    stream = torch.cuda.current_stream(device).cuda_stream
    data = torch.empty(npages * spec.page_bytes, dtype=torch.uint8, device=device)
    lines = torch.zeros(npages, dtype=torch.int32, device=device)
    rc = L.bmrg_dev_pages(C.byref(P), page0, npages, data.data_ptr(), lines.data_ptr(), stream)
    if rc:
        raise RuntimeError(f"bmrg_dev_pages rc={rc}")
    lines64 = lines.to(torch.int64)
    base = torch.zeros(npages, dtype=torch.int64, device=device)
    if npages > 1:
        base[1:] = torch.cumsum(lines64, 0)[:-1]
    n = int(lines64.sum().item())
    offsets = torch.empty(n + 1, dtype=torch.int64, device=device)
    rc = L.bmrg_dev_offsets(data.data_ptr(), npages, spec.page_bytes, base.data_ptr(), offsets.data_ptr(), stream)
    if rc:
        raise RuntimeError(f"bmrg_dev_offsets rc={rc}")
    torch.cuda.synchronize(device)
    del dt
    return {"data": data, "offsets": offsets, "n": n, "base": page0 * spec.page_bytes}


def device_km(spec: KMSpec, n: int, i0: int = 0, device: str = "cuda"):
    import torch
    c, _ = km_centres(spec)
    cd = torch.from_numpy(c.reshape(-1)).to(device)
    out = torch.empty((n, KM_DIM), dtype=torch.float32, device=device)
    rc = _clib().bmrg_dev_km(spec.seed & 0xFFFFFFFFFFFFFFFF, i0, n, cd.data_ptr(), spec.k, out.data_ptr(),
                             torch.cuda.current_stream(device).cuda_stream)
    if rc:
        raise RuntimeError(f"bmrg_dev_km rc={rc}")
    torch.cuda.synchronize(device)
    return out
