"""paper_conf_ipps_jim11_b200 — thin Python binding of libbmr (include/bmr.h).

Argument marshalling only: every step of Map -> group-by-key -> Reduce runs in the CUDA
kernels of ``libbmr.so`` (sm_100a).  PyTorch is used by callers for device memory and streams;
this module accepts torch CUDA tensors (or raw device pointers) and numpy arrays for the host
entry point.  There is no CPU fallback: if ``libbmr.so`` is missing or no CUDA device is
present, calls raise.

Names follow the C ABI: ``Job.map`` = ``mr_map``, ``Job.group`` = ``mr_group``, ...
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("BMR_LIB") or os.path.join(_HERE, "libbmr.so")   # BMR_LIB: variant builds (sweeps)

MR_ABI_VERSION = 1
WORDCOUNT, STRINGMATCH, KMEANS, INVINDEX = 1, 2, 3, 4
WORKLOADS = {"wc": WORDCOUNT, "sm": STRINGMATCH, "km": KMEANS, "ii": INVINDEX}
FLAG_NO_SMEM_IN, FLAG_NO_SMEM_OUT, FLAG_FORCE_TINY_OUT = 0x01, 0x02, 0x04
FLAG_WEAK_HASH_DEBUG, FLAG_VALIDATE, FLAG_NO_COMBINE = 0x08, 0x10, 0x20
FLAG_PROFILE, FLAG_OWN_STREAM, FLAG_NO_MAP_COMBINE, FLAG_SM_LINES = 0x40, 0x80, 0x100, 0x200
FLAG_BATCH_COMBINE, FLAG_FORCE_SPILL, FLAG_KM_FULL_SCAN = 0x400, 0x800, 0x1000

STATUS = {0: "MR_OK", 1: "MR_ERR_INVALID", 2: "MR_ERR_STATE", 3: "MR_ERR_OOM", 4: "MR_ERR_OVERFLOW",
          5: "MR_ERR_CUDA", 6: "MR_ERR_NCCL", 7: "MR_ERR_UNSUPPORTED"}

EXPORTS = ("mr_job_create", "mr_map", "mr_map_host", "mr_map_host_lines", "mr_group", "mr_reduce", "mr_fetch", "mr_job_reset",
           "mr_get_stats", "mr_job_destroy", "mr_status_string", "mr_last_error", "mr_sort_u64",
           "mr_partition_count", "mr_partition_write", "mr_ingest", "mr_set_xwindows", "mr_ingest_xwindow",
           "mr_dev_alloc", "mr_dev_free", "mr_dev_zero", "mr_dev_copy", "mr_ipc_handle", "mr_ipc_open", "mr_ipc_close",
           "mr_comm_unique_id", "mr_comm_init", "mr_comm_destroy", "mr_comm_backend")
MR_NCCL_ID_BYTES = 128


class XWindow:
    """A receive window of the fused Map flush (f-3): entry_cap 16-byte entries, heap_cap key bytes
    and the 2 x u64 cursor.  ipc=False: torch tensors on `device` (same-process ranks); ipc=True:
    one mr_dev_alloc block [cursor | entries | heap] whose CUDA IPC handle other processes open
    (XWindow.open_peer), so their Maps store into it over NVLink."""

    _HDR = 256

    def __init__(self, entry_cap: int, heap_cap: int, device=None, ipc: bool = False):
        import torch
        dev = device if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.entry_cap, self.heap_cap = int(entry_cap), int(heap_cap)
        self.ipc, self.peer, self._base = ipc, False, 0
        if not ipc:
            self.entries = torch.empty(max(self.entry_cap, 1) * 16, dtype=torch.uint8, device=dev)
            self.heap = torch.empty(max(self.heap_cap, 8), dtype=torch.uint8, device=dev)
            self.cursor = torch.zeros(2, dtype=torch.int64, device=dev)
            self.entries_ptr, self.heap_ptr = self.entries.data_ptr(), self.heap.data_ptr()
            self.cursor_ptr = self.cursor.data_ptr()
            return
        self.device = dev.index if dev.index is not None else torch.cuda.current_device()
        p = C.c_void_p()
        st = lib().mr_dev_alloc(self.device, self._bytes(), C.byref(p))
        if st:
            raise MRError(st, "mr_dev_alloc")
        self._base = p.value
        self._set_ptrs(self._base)
        self.reset()

    def _bytes(self):
        return self._HDR + max(self.entry_cap, 1) * 16 + ((max(self.heap_cap, 8) + 255) // 256) * 256

    def _set_ptrs(self, base):
        self.cursor_ptr = base
        self.entries_ptr = base + self._HDR
        self.heap_ptr = base + self._HDR + max(self.entry_cap, 1) * 16

    def ipc_handle(self) -> bytes:
        """(handle bytes, entry_cap, heap_cap) for another process to open this window."""
        h = C.create_string_buffer(64)
        st = lib().mr_ipc_handle(self._base, h)
        if st:
            raise MRError(st, "mr_ipc_handle")
        return h.raw

    @classmethod
    def open_peer(cls, handle: bytes, entry_cap: int, heap_cap: int, device: int):
        """Map another process's window (its ipc_handle) into this process."""
        w = cls.__new__(cls)
        w.entry_cap, w.heap_cap, w.ipc, w.peer, w.device = int(entry_cap), int(heap_cap), True, True, device
        p = C.c_void_p()
        st = lib().mr_ipc_open(device, C.create_string_buffer(handle, 64), C.byref(p))
        if st:
            raise MRError(st, "mr_ipc_open")
        w._base = p.value
        w._set_ptrs(w._base)
        return w

    def reset(self):
        if self.ipc:
            st = lib().mr_dev_zero(self.cursor_ptr, 16)
            if st:
                raise MRError(st, "mr_dev_zero")
        else:
            self.cursor.zero_()

    def used(self):
        """(entries, heap bytes) appended so far (demand; may exceed the capacity)."""
        c = np.zeros(2, np.uint64)
        st = lib().mr_dev_copy(c.ctypes.data, self.cursor_ptr, 16)
        if st:
            raise MRError(st, "mr_dev_copy")
        return int(c[0]), int(c[1])

    def close(self):
        if self.ipc and self._base:
            (lib().mr_ipc_close if self.peer else lib().mr_dev_free)(self._base)
            self._base = 0


class MRError(RuntimeError):
    def __init__(self, status: int, detail: str = ""):
        self.status = status
        super().__init__(f"{STATUS.get(status, status)}: {detail}")


class Config(C.Structure):
    _fields_ = [("abi_version", C.c_uint32), ("workload", C.c_int), ("device", C.c_int), ("stream", C.c_void_p),
                ("record_stride", C.c_uint32), ("params", C.c_void_p), ("input_base", C.c_uint64),
                ("rank", C.c_int), ("nranks", C.c_int), ("nccl_comm", C.c_void_p),
                ("max_pairs_hint", C.c_uint64), ("heap_bytes_hint", C.c_uint64), ("flags", C.c_uint32)]


class SMParams(C.Structure):
    _fields_ = [("pattern", C.c_uint8 * 16)]


class KMParams(C.Structure):
    _fields_ = [("k", C.c_uint32), ("dim", C.c_uint32), ("centroids", C.c_void_p)]


class Result(C.Structure):
    _fields_ = [("n_keys", C.c_uint64), ("keys", C.c_void_p), ("key_offsets", C.c_void_p),
                ("vals", C.c_void_p), ("val_offsets", C.c_void_p)]


class Stats(C.Structure):
    _fields_ = [(n, C.c_uint64) for n in ("pairs", "flushes", "replays", "n_keys", "collisions", "sort_passes",
                                          "map_tiles", "input_bytes", "capacity_pairs", "kernel_launches")] + \
               [(n, C.c_double) for n in ("map_ms", "hist_ms", "sort_ms", "seg_ms", "reduce_ms")] + \
               [("pairs_hashed", C.c_uint64), ("sort_passes_keys", C.c_uint64), ("sort_keys_ms", C.c_double),
                ("pairs_mid", C.c_uint64), ("sort_passes_mid", C.c_uint64),
                ("pairs_partial", C.c_uint64), ("words_combined", C.c_uint64),
                ("xchg_send_bytes", C.c_uint64), ("xchg_recv_bytes", C.c_uint64), ("xchg_ms", C.c_double),
                ("map_seal_waits", C.c_uint64), ("map_spills", C.c_uint64),
                ("km_points_scanned", C.c_uint64)]


_LIB = None


def lib() -> C.CDLL:
    """Load libbmr.so (fails loudly if it was not built)."""
    global _LIB
    if _LIB is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} not built: run __graft_entry__.build()")
        if "BMR_NCCL_LIB" not in os.environ:   # the NCCL torch bundles (libbmr dlopens it for mr_group's exchange)
            try:
                import nvidia.nccl
                cand = os.path.join(list(nvidia.nccl.__path__)[0], "lib", "libnccl.so.2")
                if os.path.exists(cand):
                    os.environ["BMR_NCCL_LIB"] = cand
            except ImportError:
                pass
        L = C.CDLL(LIB_PATH)
        vp, u64 = C.c_void_p, C.c_uint64
        L.mr_job_create.argtypes = [C.POINTER(Config), C.POINTER(vp)]
        L.mr_map.argtypes = [vp, vp, vp, u64]
        L.mr_map_host.argtypes = [vp, vp, vp, u64]
        L.mr_map_host_lines.argtypes = [vp, vp, u64]
        for f in ("mr_group", "mr_reduce", "mr_job_reset", "mr_job_destroy"):
            getattr(L, f).argtypes = [vp]
        L.mr_fetch.argtypes = [vp, C.POINTER(Result)]
        L.mr_get_stats.argtypes = [vp, vp, C.c_size_t]
        L.mr_status_string.argtypes = [C.c_int]
        L.mr_status_string.restype = C.c_char_p
        L.mr_last_error.argtypes = [vp]
        L.mr_last_error.restype = C.c_char_p
        L.mr_sort_u64.argtypes = [vp, vp, vp, u64, vp]
        L.mr_partition_count.argtypes = [vp, vp, C.POINTER(u64)]
        L.mr_partition_write.argtypes = [vp, vp, vp]
        L.mr_ingest.argtypes = [vp, vp, vp, vp]
        L.mr_set_xwindows.argtypes = [vp, C.c_uint32, vp, vp, vp, u64, u64]
        L.mr_ingest_xwindow.argtypes = [vp, vp, vp, vp, u64, u64]
        L.mr_dev_alloc.argtypes = [C.c_int, u64, vp]
        L.mr_dev_free.argtypes = [vp]
        L.mr_dev_zero.argtypes = [vp, u64]
        L.mr_dev_copy.argtypes = [vp, vp, u64]
        L.mr_ipc_handle.argtypes = [vp, vp]
        L.mr_ipc_open.argtypes = [C.c_int, vp, vp]
        L.mr_ipc_close.argtypes = [vp]
        L.mr_comm_unique_id.argtypes = [vp]
        L.mr_comm_init.argtypes = [vp, C.c_int, C.c_int, C.c_int, C.POINTER(vp)]
        L.mr_comm_destroy.argtypes = [vp]
        L.mr_comm_backend.argtypes = []
        L.mr_comm_backend.restype = C.c_char_p
        for f in EXPORTS:
            if f not in ("mr_status_string", "mr_last_error", "mr_comm_backend"):
                getattr(L, f).restype = C.c_int
        _LIB = L
    return _LIB


def _ptr(x) -> int:
    if x is None:
        return 0
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return int(x.data_ptr())
    if isinstance(x, np.ndarray):
        return int(x.ctypes.data)
    raise TypeError(type(x))


def _copy(addr, nbytes, dtype=np.uint8, copy=True):
    if nbytes == 0:
        return np.zeros(0, dtype)
    a = np.frombuffer((C.c_uint8 * nbytes).from_address(addr), np.uint8)
    return (a.copy() if copy else a).view(dtype)


class Comm:
    """An NCCL communicator created by libbmr (mr_comm_unique_id / mr_comm_init) for the exchange
    inside mr_group: ``Job(..., comm=c)``.  ``Comm.from_torch()`` forms it over the default
    torch.distributed group (the 128-byte id travels by broadcast_object_list: plumbing only)."""

    def __init__(self, uid: bytes, nranks: int, rank: int, device: int):
        p = C.c_void_p()
        st = lib().mr_comm_init(C.create_string_buffer(uid, MR_NCCL_ID_BYTES), nranks, rank, device, C.byref(p))
        if st:
            raise MRError(st, f"mr_comm_init ({lib().mr_comm_backend().decode()})")
        self.ptr, self.nranks, self.rank, self.device = p.value, nranks, rank, device

    @staticmethod
    def unique_id() -> bytes:
        b = C.create_string_buffer(MR_NCCL_ID_BYTES)
        st = lib().mr_comm_unique_id(b)
        if st:
            raise MRError(st, f"mr_comm_unique_id ({lib().mr_comm_backend().decode()})")
        return b.raw

    @classmethod
    def from_torch(cls, group=None, device: int | None = None):
        import torch
        import torch.distributed as dist
        rank, world = dist.get_rank(group), dist.get_world_size(group)
        obj = [cls.unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=dist.get_global_rank(group, 0) if group is not None else 0, group=group)
        return cls(obj[0], world, rank, torch.cuda.current_device() if device is None else device)

    @staticmethod
    def backend() -> str:
        return lib().mr_comm_backend().decode()

    def close(self):
        if getattr(self, "ptr", None):
            lib().mr_comm_destroy(self.ptr)
            self.ptr = None


class Job:
    """One MapReduce job (mr_job).  ``workload`` in {"wc", "sm", "km", "ii"}.  With ``comm`` (a
    Comm over ``nranks`` processes) mr_group performs the multi-GPU exchange itself."""

    def __init__(self, workload: str, device: int = 0, stream=None, pattern: bytes | None = None,
                 centroids: np.ndarray | None = None, input_base: int = 0, flags: int = 0,
                 max_pairs_hint: int = 0, rank: int = 0, nranks: int = 1, comm: Comm | None = None):
        L = lib()
        self.workload = workload
        cfg = Config()
        cfg.abi_version = MR_ABI_VERSION
        cfg.workload = WORKLOADS[workload]
        cfg.device = device
        if stream is None:
            import torch
            stream = torch.cuda.current_stream(device).cuda_stream
        cfg.stream = stream
        cfg.input_base = input_base
        cfg.rank, cfg.nranks = rank, nranks
        self.rank, self.nranks = rank, nranks
        if comm is not None:
            assert comm.nranks == nranks and comm.rank == rank, "comm does not match (rank, nranks)"
            cfg.nccl_comm = comm.ptr
        self.comm = comm
        cfg.max_pairs_hint = max_pairs_hint
        cfg.flags = flags
        self._keep = []
        if workload == "sm":
            p = SMParams()
            for i, b in enumerate(pattern[:16]):
                p.pattern[i] = b
            cfg.params = C.addressof(p)
            self._keep.append(p)
        elif workload == "km":
            cen = np.ascontiguousarray(centroids, np.float32)
            p = KMParams(cen.shape[0], cen.shape[1], cen.ctypes.data)
            cfg.params = C.addressof(p)
            cfg.record_stride = 32
            self._keep += [p, cen]
        h = C.c_void_p()
        self._check(L.mr_job_create(C.byref(cfg), C.byref(h)), None)
        self.h = h

    def _check(self, rc, h=-1):
        if rc != 0:
            hh = self.h if h == -1 else h
            detail = lib().mr_last_error(hh).decode() if hh else ""
            raise MRError(rc, detail)

    def map(self, records, offsets=None, n: int | None = None):
        """mr_map over device records (torch uint8 CUDA tensor or pointer); offsets: int64 tensor
        holding the n+1 u64 offsets (None for KM)."""
        if n is None:
            n = (offsets.numel() - 1) if offsets is not None else records.numel() // 32
        self._check(lib().mr_map(self.h, _ptr(records), _ptr(offsets), n))

    def map_host(self, records: np.ndarray, offsets: np.ndarray | None = None, n: int | None = None):
        if n is None:
            n = (len(offsets) - 1) if offsets is not None else records.size // 32
        self._check(lib().mr_map_host(self.h, _ptr(records), _ptr(offsets), n))

    def map_host_lines(self, text: np.ndarray):
        """Host text whose records are its '\n'-terminated lines (offsets derived on the device,
        copies overlapped with the Map; pin `text` for the overlap)."""
        self._check(lib().mr_map_host_lines(self.h, _ptr(text), int(text.size)))

    def group(self):
        self._check(lib().mr_group(self.h))

    def reduce(self):
        self._check(lib().mr_reduce(self.h))

    def fetch(self, copy: bool = True) -> dict:
        """The result (mr_result encoding).  copy=False returns views of the job-owned pinned host
        buffers (valid until the next call on this job, as in the C ABI)."""
        r = Result()
        self._check(lib().mr_fetch(self.h, C.byref(r)))
        n = int(r.n_keys)
        ko = _copy(r.key_offsets, 8 * (n + 1), np.uint64, copy)
        vo = _copy(r.val_offsets, 8 * (n + 1), np.uint64, copy)
        return {"n_keys": n, "keys": _copy(r.keys, int(ko[-1]), np.uint8, copy), "key_offsets": ko,
                "vals": _copy(r.vals, int(vo[-1]), np.uint8, copy), "val_offsets": vo}

    def run(self, *batches) -> dict:
        for b in batches:
            self.map(*b)
        self.group()
        self.reduce()
        return self.fetch()

    # ---- multi-GPU exchange (mr_partition_count / mr_partition_write / mr_ingest) ----
    def partition(self):
        """Partition this rank's records by destination; returns (entries u8 tensor, heap u8
        tensor, counts int64 array [nranks, 2] = (entries, heap bytes) per destination, entry_bytes)."""
        import torch
        counts = np.zeros(2 * self.nranks, np.uint64)
        eb = C.c_uint64(0)
        self._check(lib().mr_partition_count(self.h, _ptr(counts), C.byref(eb)))
        counts = counts.astype(np.int64).reshape(self.nranks, 2)
        dev = torch.device("cuda", torch.cuda.current_device())
        ent = torch.empty(int(counts[:, 0].sum()) * eb.value, dtype=torch.uint8, device=dev)
        heap = torch.empty(int(counts[:, 1].sum()), dtype=torch.uint8, device=dev)
        self._check(lib().mr_partition_write(self.h, _ptr(ent), _ptr(heap)))
        return ent, heap, counts, int(eb.value)

    def ingest(self, entries, heap, recv_counts):
        """mr_ingest of the buffers received from every source rank (concatenated in rank order);
        recv_counts int64 [nranks, 2].  The buffers must stay alive until reduce completes."""
        rc = np.ascontiguousarray(recv_counts, np.int64).astype(np.uint64).reshape(-1)
        self._recv = (entries, heap, rc)
        self._check(lib().mr_ingest(self.h, _ptr(entries), _ptr(heap), _ptr(rc)))

    # ---- fused Map flush + shuffle (mr_set_xwindows / mr_ingest_xwindow) ----
    def set_xwindows(self, windows):
        """Register one receive window per destination rank (list of XWindow, rank order) before
        map(): InvertedIndex records then leave the Map straight through them."""
        n = len(windows)
        arr = (C.c_void_p * max(n, 1))
        ents = arr(*[w.entries_ptr for w in windows])
        heaps = arr(*[w.heap_ptr for w in windows])
        curs = arr(*[w.cursor_ptr for w in windows])
        ecap = windows[0].entry_cap if n else 0
        hcap = windows[0].heap_cap if n else 0
        self._xwin = list(windows)
        self._check(lib().mr_set_xwindows(self.h, n, C.cast(ents, C.c_void_p), C.cast(heaps, C.c_void_p),
                                          C.cast(curs, C.c_void_p), ecap, hcap))

    def ingest_xwindow(self, w):
        """Ingest this rank's own receive window after every rank's Map completed."""
        self._recv = (w,)
        self._check(lib().mr_ingest_xwindow(self.h, w.entries_ptr, w.heap_ptr, w.cursor_ptr, w.entry_cap, w.heap_cap))

    def shuffle(self, group=None):
        """One all-to-all exchange over torch.distributed (NCCL on GPUs): partition -> exchange
        -> ingest."""
        from . import dist as D
        ent, heap, counts, eb = self.partition()
        recv_counts = D.exchange_counts(counts, group)
        r_ent = D.alltoallv(ent, counts[:, 0] * eb, recv_counts[:, 0] * eb, group)
        r_heap = D.alltoallv(heap, counts[:, 1], recv_counts[:, 1], group)
        self.ingest(r_ent, r_heap, recv_counts)
        return int(counts[:, 0].sum()) * eb + int(counts[:, 1].sum())

    def reset(self):
        self._check(lib().mr_job_reset(self.h))

    def stats(self) -> dict:
        s = Stats()
        self._check(lib().mr_get_stats(self.h, C.byref(s), C.sizeof(s)))
        return {n: (float(getattr(s, n)) if t is C.c_double else int(getattr(s, n))) for n, t in Stats._fields_}

    def close(self):
        if getattr(self, "h", None):
            lib().mr_job_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


def sort_u64(keys, stream=None):
    """mr_sort_u64 on an int64 CUDA tensor (u64 bit patterns): returns (sorted keys, perm int32)."""
    import torch
    n = keys.numel()
    out = torch.empty_like(keys)
    perm = torch.empty(n, dtype=torch.int32, device=keys.device)
    if stream is None:
        stream = torch.cuda.current_stream(keys.device).cuda_stream
    rc = lib().mr_sort_u64(_ptr(keys), _ptr(out), _ptr(perm), n, stream)
    if rc:
        raise MRError(rc, "mr_sort_u64")
    return out, perm
