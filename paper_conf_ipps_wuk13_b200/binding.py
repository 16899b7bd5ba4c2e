"""ctypes binding of libshingle.so (include/shingle.h) — argument marshalling only.

Every step of the hot path runs in the library's CUDA kernels; this module
never computes any part of the method and has no CPU fallback: if the shared
library or a CUDA device is missing, the calls raise.
Function names mirror the C ABI one to one.
"""
from __future__ import annotations

import ctypes as C
import os
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# SG_LIB: test / A-B hook to load another build of the same library
LIB_PATH = os.environ.get("SG_LIB") or os.path.join(_HERE, "libshingle.so")

SG_OK, SG_EINVAL, SG_ENOMEM, SG_ESTATE, SG_ECUDA, SG_ENCCL, SG_EOVERFLOW = range(7)
SG_DEVICE_PTRS = 0x1
SG_NO_VALIDATE = 0x2
SG_HOST_CSR = 0x4
STATUS_NAMES = {0: "SG_OK", 1: "SG_EINVAL", 2: "SG_ENOMEM", 3: "SG_ESTATE", 4: "SG_ECUDA",
                5: "SG_ENCCL", 6: "SG_EOVERFLOW"}
STAGES = ["pass1", "group1", "pass2", "group2", "select1", "hash1", "select2", "hash2",
          "hist1", "scatter1", "local1", "hist2", "scatter2", "local2", "exchange1", "exchange2",
          "fine1", "fine2", "report"]
SG_REPORT_HOST = 0x10


class SGError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


class sg_dist(C.Structure):
    _fields_ = [("rank", C.c_int32), ("world", C.c_int32), ("device", C.c_int32),
                ("stream", C.c_void_p), ("nccl_uid", C.c_void_p), ("loopback", C.c_void_p),
                ("flags", C.c_uint32)]


SG_DIST_EXCHANGE = 0x1
SG_DIST_PEER = 0x2


_lib = None


def lib() -> C.CDLL:
    """Load libshingle.so (built by __graft_entry__.build()).  Raises if absent."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built: run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = C.CDLL(LIB_PATH)
    i32, i64, u32, u64, vp = C.c_int32, C.c_int64, C.c_uint32, C.c_uint64, C.c_void_p
    st = C.c_int
    sig = {
        "shingle_graph_create": (st, [i64, i64, vp, vp, u32, vp, C.POINTER(vp)]),
        "shingle_graph_load": (st, [vp, i64, i64, vp, vp, u32]),
        "shingle_pass": (st, [vp, i32, i32, u64]),
        "group_by_shingle": (st, [vp]),
        "report_dense_subgraphs": (st, [vp, i32, i32, vp, vp]),
        "report_overlapping_clusters": (st, [vp, i32, i32, vp, vp, vp, vp]),
        "sg_cluster_density": (st, [vp, vp, i32, vp, vp, vp]),
        "sg_partition_agreement": (st, [vp, vp, vp, vp]),
        "sg_connected_components": (st, [vp, vp, vp]),
        "shingle_graph_reset": (st, [vp]),
        "shingle_graph_destroy": (None, [vp]),
        "sg_last_error": (C.c_char_p, [vp]),
        "sg_get_counts": (st, [vp, vp]),
        "sg_get_shingles": (st, [vp, i32, vp, vp, i64, vp, vp]),
        "sg_get_groups": (st, [vp, i32, vp, vp, vp, vp, vp, vp]),
        "sg_get_groups_range": (st, [vp, i32, i32, i32, vp, vp, vp, vp, vp, vp]),
        "sg_get_shingles_range": (st, [vp, i32, i32, i32, vp, vp, i64, vp, vp]),
        "sg_get_s1p": (st, [vp, vp, i64, vp, vp]),
        "sg_get_hash_params": (st, [vp, i32, vp, vp, i32]),
        "sg_get_stage_ms": (st, [vp, vp, i32, vp]),
        "sg_loopback_create": (st, [i32, C.POINTER(vp)]),
        "sg_loopback_destroy": (None, [vp]),
        "sg_partition_rows": (st, [i64, vp, i32, i64, vp]),
        "sg_nccl_unique_id": (st, [vp]),
        "sg_s1p_offsets": (st, [i32, i32, i32, vp, vp, vp, vp]),
        "sg_version": (C.c_char_p, []),
        "sg_component_shards": (st, [i64, vp, vp, i32, i64, vp, vp]),
        "sg_shard_csr": (st, [i64, vp, vp, vp, i32, vp, vp, vp]),
        "sg_merge_shard_labels": (st, [i64, vp, i32, vp, vp]),
    }
    for name, (rt, args) in sig.items():
        f = getattr(L, name)
        f.restype = rt
        f.argtypes = args
    _lib = L
    return L


def _check(rc: int, h=None):
    if rc != SG_OK:
        msg = lib().sg_last_error(h)
        raise SGError(rc, msg.decode() if msg else "")


def _addr(x) -> int:
    """Data address of a numpy array or a torch tensor."""
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    return x.data_ptr()


def _is_cuda(x) -> bool:
    return hasattr(x, "is_cuda") and x.is_cuda


# ------------------------------------------------------------------ C ABI calls
def shingle_graph_create(row_ptr, col, validate: bool = True, dist: Optional[dict] = None,
                         host_csr: bool = False):
    """row_ptr int64[n+1], col int32[nnz]: numpy arrays (host) or CUDA tensors.
    host_csr: out-of-core entries (col stays in host memory, mapped; keep the
    array alive and unchanged while the handle uses it)."""
    dev = _is_cuda(row_ptr)
    if not dev:
        row_ptr = np.ascontiguousarray(row_ptr, np.int64)
        col = np.ascontiguousarray(col, np.int32)
    n = int(row_ptr.shape[0]) - 1
    nnz = int(col.shape[0])
    flags = (SG_DEVICE_PTRS if dev else 0) | (0 if validate else SG_NO_VALIDATE) | \
        (SG_HOST_CSR if host_csr else 0)
    dptr = None
    if dist is not None:
        d = sg_dist(int(dist.get("rank", 0)), int(dist.get("world", 1)), int(dist.get("device", 0)),
                    dist.get("stream"), None, dist.get("loopback"),
                    (SG_DIST_EXCHANGE if dist.get("exchange") else 0) |
                    (SG_DIST_PEER if dist.get("peer") else 0))
        uid = dist.get("nccl_uid")
        if uid is not None:
            d._uid_buf = C.create_string_buffer(bytes(uid), 128)
            d.nccl_uid = C.cast(d._uid_buf, C.c_void_p)
        dptr = C.byref(d)
    out = C.c_void_p()
    rc = lib().shingle_graph_create(n, nnz, _addr(row_ptr), _addr(col), flags, dptr, C.byref(out))
    _check(rc)
    return out


def shingle_graph_load(h, row_ptr, col, validate: bool = True, host_csr: bool = False):
    """Replace the resident graph of handle h (host arrays or CUDA tensors)."""
    dev = _is_cuda(row_ptr)
    if not dev:
        row_ptr = np.ascontiguousarray(row_ptr, np.int64)
        col = np.ascontiguousarray(col, np.int32)
    n = int(row_ptr.shape[0]) - 1
    flags = (SG_DEVICE_PTRS if dev else 0) | (0 if validate else SG_NO_VALIDATE) | \
        (SG_HOST_CSR if host_csr else 0)
    _check(lib().shingle_graph_load(h, n, int(col.shape[0]), _addr(row_ptr), _addr(col), flags), h)


def _labels_arg(h, labels, what="labels"):
    """int32 label array of exactly n entries (the C side reads n values)."""
    a = np.ascontiguousarray(labels, np.int32)
    n = sg_get_counts(h)["n"]
    if a.ndim != 1 or len(a) != n:
        raise ValueError(f"{what} must have n = {n} entries (got shape {a.shape})")
    return a


def shingle_pass(h, s: int, c: int, seed: int):
    _check(lib().shingle_pass(h, s, c, seed & 0xFFFFFFFFFFFFFFFF), h)


def group_by_shingle(h):
    _check(lib().group_by_shingle(h), h)


def report_dense_subgraphs(h, mode: int = 0, min_size: int = 1, n: Optional[int] = None):
    if n is None:
        n = sg_get_counts(h)["n"]
    labels = np.zeros(n, np.int32)
    nc = C.c_int64()
    _check(lib().report_dense_subgraphs(h, mode, min_size, labels.ctypes.data, C.byref(nc)), h)
    return labels, nc.value


def report_overlapping_clusters(h, mode: int = 0, min_size: int = 1):
    """Phase III approach 1: (offs int64[C+1], verts uint32[V])."""
    cnt = np.zeros(2, np.int64)
    _check(lib().report_overlapping_clusters(h, mode, min_size, None, None, None, cnt.ctypes.data), h)
    offs = np.zeros(int(cnt[0]) + 1, np.int64)
    verts = np.zeros(int(cnt[1]), np.uint32)
    caps = np.array([len(offs), len(verts)], np.int64)
    _check(lib().report_overlapping_clusters(h, mode, min_size, offs.ctypes.data, verts.ctypes.data,
                                             caps.ctypes.data, cnt.ctypes.data), h)
    return offs, verts


def sg_cluster_density(h, labels, min_size: int = 2):
    """Eq. 6 density over the clusters of `labels`: (mean, stddev, n_clusters)."""
    labels = _labels_arg(h, labels)
    mean, sd, nc = C.c_double(), C.c_double(), C.c_int64()
    _check(lib().sg_cluster_density(h, labels.ctypes.data, min_size, C.byref(mean), C.byref(sd),
                                    C.byref(nc)), h)
    return mean.value, sd.value, nc.value


def sg_partition_agreement(h, test_labels, bench_labels) -> dict:
    """Pair counts TP, FP, FN, TN and Eq. 2-5 (PPV, NPV, SP, SE)."""
    t = _labels_arg(h, test_labels, "test_labels")
    b = _labels_arg(h, bench_labels, "bench_labels")
    cnt = np.zeros(4, np.int64)
    _check(lib().sg_partition_agreement(h, t.ctypes.data, b.ctypes.data, cnt.ctypes.data), h)
    tp, fp, fn, tn = (int(x) for x in cnt)

    def ratio(a, b):
        return a / b if b else float("nan")
    return dict(TP=tp, FP=fp, FN=fn, TN=tn, PPV=ratio(tp, tp + fp), NPV=ratio(tn, tn + fn),
                SP=ratio(tn, tn + fp), SE=ratio(tp, tp + fn))


def sg_connected_components(h, n: Optional[int] = None):
    """Connected components of G: (labels int32[n] = smallest vertex, count)."""
    if n is None:
        n = sg_get_counts(h)["n"]
    labels = np.zeros(n, np.int32)
    nc = C.c_int64()
    _check(lib().sg_connected_components(h, labels.ctypes.data, C.byref(nc)), h)
    return labels, nc.value


def shingle_graph_reset(h):
    _check(lib().shingle_graph_reset(h), h)


def shingle_graph_destroy(h):
    lib().shingle_graph_destroy(h)


def sg_get_counts(h) -> dict:
    a = np.zeros(16, np.int64)
    _check(lib().sg_get_counts(h, a.ctypes.data), h)
    keys = ["n", "row_lo", "rows", "n_e", "groups1", "s1p", "groups2", "pairs1", "pairs2", "state",
            "entries2", "launches", "chunks1", "chunks2", "world", "exchange"]
    return dict(zip(keys, (int(x) for x in a)))


def sg_get_shingles(h, level: int):
    rows, c = C.c_int64(), C.c_int32()
    _check(lib().sg_get_shingles(h, level, None, None, 0, C.byref(rows), C.byref(c)), h)
    ids = np.zeros((rows.value, c.value), np.uint64)
    rowid = np.zeros(rows.value, np.uint32)
    _check(lib().sg_get_shingles(h, level, ids.ctypes.data, rowid.ctypes.data, rows.value,
                                 C.byref(rows), C.byref(c)), h)
    return ids, rowid


def sg_get_groups(h, level: int, with_ids: bool = True):
    cnt = np.zeros(3, np.int64)
    _check(lib().sg_get_groups(h, level, None, None, None, None, None, cnt.ctypes.data), h)
    G, npairs, c = (int(x) for x in cnt)
    tg = np.zeros(c + 1, np.int64)
    ids = np.zeros(G, np.uint64)
    offs = np.zeros(G + 1, np.int64)
    mem = np.zeros(npairs, np.uint32)
    caps = np.array([G, npairs], np.int64)
    _check(lib().sg_get_groups(h, level, tg.ctypes.data, ids.ctypes.data if with_ids else None,
                               offs.ctypes.data, mem.ctypes.data, caps.ctypes.data,
                               cnt.ctypes.data), h)
    return tg, (ids if with_ids else None), offs, mem


def sg_get_groups_range(h, level: int, t0: int, t1: int, with_ids: bool = True):
    """Groups of trials [t0, t1) of a level; offsets relative to trial t0."""
    cnt = np.zeros(3, np.int64)
    _check(lib().sg_get_groups_range(h, level, t0, t1, None, None, None, None, None,
                                     cnt.ctypes.data), h)
    G, npairs, nt = (int(x) for x in cnt)
    tg = np.zeros(nt + 1, np.int64)
    ids = np.zeros(G, np.uint64)
    offs = np.zeros(G + 1, np.int64)
    mem = np.zeros(npairs, np.uint32)
    caps = np.array([G, npairs], np.int64)
    _check(lib().sg_get_groups_range(h, level, t0, t1, tg.ctypes.data,
                                     ids.ctypes.data if with_ids else None, offs.ctypes.data,
                                     mem.ctypes.data, caps.ctypes.data, cnt.ctypes.data), h)
    return tg, (ids if with_ids else None), offs, mem


def sg_get_shingles_range(h, level: int, t0: int, t1: int):
    """Columns [t0, t1) of the shingle matrix: (ids[rows, t1-t0], rowid[rows])."""
    rows, c = C.c_int64(), C.c_int32()
    _check(lib().sg_get_shingles_range(h, level, t0, t1, None, None, 0, C.byref(rows), C.byref(c)), h)
    ids = np.zeros((rows.value, t1 - t0), np.uint64)
    rowid = np.zeros(rows.value, np.uint32)
    _check(lib().sg_get_shingles_range(h, level, t0, t1, ids.ctypes.data, rowid.ctypes.data,
                                       rows.value, C.byref(rows), C.byref(c)), h)
    return ids, rowid


def sg_get_s1p(h):
    cnt, k0 = C.c_int64(), C.c_int64()
    _check(lib().sg_get_s1p(h, None, 0, C.byref(cnt), C.byref(k0)), h)
    out = np.zeros(cnt.value, np.int64)
    _check(lib().sg_get_s1p(h, out.ctypes.data, cnt.value, C.byref(cnt), C.byref(k0)), h)
    return out, k0.value


def sg_get_hash_params(h, level: int, c: int):
    A = np.zeros(c, np.uint32)
    B = np.zeros(c, np.uint32)
    _check(lib().sg_get_hash_params(h, level, A.ctypes.data, B.ctypes.data, c), h)
    return A, B


def sg_get_stage_ms(h) -> dict:
    ms = np.zeros(len(STAGES), np.float32)
    n = C.c_int32()
    _check(lib().sg_get_stage_ms(h, ms.ctypes.data, len(STAGES), C.byref(n)), h)
    return {k: float(v) for k, v in zip(STAGES, ms[: n.value])}


def sg_partition_rows(row_ptr, world: int, kappa: int = 8) -> np.ndarray:
    row_ptr = np.ascontiguousarray(row_ptr, np.int64)
    b = np.zeros(world + 1, np.int64)
    _check(lib().sg_partition_rows(len(row_ptr) - 1, row_ptr.ctypes.data, world, kappa, b.ctypes.data))
    return b


def sg_loopback_create(world: int):
    out = C.c_void_p()
    _check(lib().sg_loopback_create(world, C.byref(out)))
    return out


def sg_loopback_destroy(lb):
    lib().sg_loopback_destroy(lb)


def sg_nccl_unique_id() -> bytes:
    """128-byte ncclUniqueId (rank 0 creates it; broadcast it to the others)."""
    buf = C.create_string_buffer(128)
    _check(lib().sg_nccl_unique_id(buf))
    return buf.raw


nccl_unique_id = sg_nccl_unique_id


def sg_s1p_offsets(all_counts, rank: int):
    """all_counts int64[world, c1] -> (first[c1+1], off[c1], total): canonical S1' index map."""
    a = np.ascontiguousarray(all_counts, np.int64)
    world, c1 = a.shape
    first = np.zeros(c1 + 1, np.int64)
    off = np.zeros(max(c1, 1), np.int64)
    tot = C.c_int64()
    _check(lib().sg_s1p_offsets(world, rank, c1, a.ctypes.data, first.ctypes.data, off.ctypes.data,
                                C.byref(tot)))
    return first, off[:c1], tot.value


def sg_component_shards(row_ptr, col, world: int, kappa: int = 8):
    """Whole connected components per shard (N3): (shard int32[n], load int64[world])."""
    row_ptr = np.ascontiguousarray(row_ptr, np.int64)
    col = np.ascontiguousarray(col, np.int32)
    n = len(row_ptr) - 1
    shard = np.zeros(n, np.int32)
    load = np.zeros(world, np.int64)
    _check(lib().sg_component_shards(n, row_ptr.ctypes.data, col.ctypes.data, world, kappa,
                                     shard.ctypes.data, load.ctypes.data))
    return shard, load


def sg_shard_csr(row_ptr, col, shard, r: int):
    """CSR of shard r over all vertex ids (other rows empty)."""
    row_ptr = np.ascontiguousarray(row_ptr, np.int64)
    col = np.ascontiguousarray(col, np.int32)
    shard = np.ascontiguousarray(shard, np.int32)
    n = len(row_ptr) - 1
    nnz = C.c_int64()
    _check(lib().sg_shard_csr(n, row_ptr.ctypes.data, col.ctypes.data, shard.ctypes.data, r, None, None,
                              C.byref(nnz)))
    rp = np.zeros(n + 1, np.int64)
    cl = np.zeros(nnz.value, np.int32)
    _check(lib().sg_shard_csr(n, row_ptr.ctypes.data, col.ctypes.data, shard.ctypes.data, r,
                              rp.ctypes.data, cl.ctypes.data, C.byref(nnz)))
    return rp, cl


def sg_merge_shard_labels(shard, labels_stacked):
    """labels_stacked int32[world, n] (each shard's report) -> int32[n]."""
    shard = np.ascontiguousarray(shard, np.int32)
    lab = np.ascontiguousarray(labels_stacked, np.int32)
    world, n = lab.shape
    out = np.zeros(n, np.int32)
    _check(lib().sg_merge_shard_labels(n, shard.ctypes.data, world, lab.ctypes.data, out.ctypes.data))
    return out


def sg_version() -> str:
    return lib().sg_version().decode()


# ------------------------------------------------------------------ convenience
class ShingleGraph:
    """RAII wrapper: create -> pass -> group -> pass -> group -> report."""

    def __init__(self, row_ptr, col, validate=True, dist=None, host_csr=False):
        self._keep = (row_ptr, col) if host_csr else None      # mapped by the handle
        self.h = shingle_graph_create(row_ptr, col, validate=validate, dist=dist, host_csr=host_csr)
        self.n = int(row_ptr.shape[0]) - 1

    def run(self, s1, c1, seed1, s2, c2, seed2):
        shingle_pass(self.h, s1, c1, seed1)
        group_by_shingle(self.h)
        shingle_pass(self.h, s2, c2, seed2)
        group_by_shingle(self.h)
        return self

    def report(self, mode=0, min_size=1):
        return report_dense_subgraphs(self.h, mode, min_size, self.n)

    def components(self):
        return sg_connected_components(self.h, self.n)

    def agreement(self, test_labels, bench_labels):
        return sg_partition_agreement(self.h, test_labels, bench_labels)

    def density(self, labels, min_size=2):
        return sg_cluster_density(self.h, labels, min_size)

    def report_overlapping(self, mode=0, min_size=1):
        return report_overlapping_clusters(self.h, mode, min_size)

    def reset(self):
        shingle_graph_reset(self.h)

    def close(self):
        if self.h is not None:
            shingle_graph_destroy(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
