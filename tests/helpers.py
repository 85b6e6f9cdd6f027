"""Test utilities: decode the mr_result encoding into canonical Python objects.

These only re-pack bytes; no MapReduce arithmetic lives here."""
from __future__ import annotations

import numpy as np


def _items(r):
    ko, vo, k, v = r["key_offsets"], r["val_offsets"], r["keys"], r["vals"]
    for i in range(int(r["n_keys"])):
        yield bytes(k[ko[i]:ko[i + 1]]), bytes(v[vo[i]:vo[i + 1]])


def decode(workload: str, r: dict):
    """Canonical form (C-1 step 4): WC {word: count}; SM sorted u64 offsets;
    KM (centroids f32[k,8], counts u64[k]) by id; II {url: tuple(sorted offsets)}."""
    if workload == "wc":
        out = {}
        for kb, vb in _items(r):
            assert kb not in out, "duplicate key"
            out[kb] = int(np.frombuffer(vb, np.uint64)[0])
        return out
    if workload == "sm":
        keys = np.frombuffer(bytes(r["keys"]), np.uint64) if r["n_keys"] else np.zeros(0, np.uint64)
        return np.sort(keys)
    if workload == "km":
        items = sorted(((int(np.frombuffer(kb, np.uint32)[0]), vb) for kb, vb in _items(r)))
        k = len(items)
        cen = np.zeros((k, 8), np.float32)
        cnt = np.zeros(k, np.uint64)
        for j, (cid, vb) in enumerate(items):
            assert cid == j
            cen[j] = np.frombuffer(vb[:32], np.float32)
            cnt[j] = np.frombuffer(vb[32:40], np.uint64)[0]
        return cen, cnt
    if workload == "ii":
        out = {}
        for kb, vb in _items(r):
            assert kb not in out, "duplicate key"
            out[kb] = tuple(sorted(np.frombuffer(vb, np.uint64).tolist()))
        return out
    raise ValueError(workload)


def split_records(data: np.ndarray, offsets: np.ndarray):
    b = bytes(data)
    return [b[int(offsets[i]):int(offsets[i + 1])] for i in range(len(offsets) - 1)]


def make_records(recs: list[bytes]):
    """records u8 + offsets u64 from a list of byte strings."""
    data = np.frombuffer(b"".join(recs), np.uint8).copy() if recs else np.zeros(0, np.uint8)
    off = np.zeros(len(recs) + 1, np.uint64)
    off[1:] = np.cumsum([len(x) for x in recs]) if recs else []
    return data, off
