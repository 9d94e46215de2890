"""B200-native lazy-update grid index (G-Grid) for snapshot kNN over moving objects.

Thin Python binding over the C ABI in include/ggrid.h (libggrid.so, built in-tree by
`paper_conf_icde_li0qhdy18_b200.build`).  Argument marshalling only: every step of
ingest / flush / expansion / top-k runs in the CUDA kernels of csrc/.  There is no CPU
fallback: if libggrid.so is missing or no CUDA device is present the calls raise.

The same names as the C ABI are exported (ggrid_build, ggrid_ingest, ggrid_knn, ...), plus
a small `GGrid` convenience class.  Arrays may be numpy arrays (host) or torch tensors
(host or CUDA); the library detects host vs device pointers itself.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("GGRID_LIB") or os.path.join(_PKG, "libggrid.so")

GGRID_OK, GGRID_EINVAL, GGRID_ENOMEM, GGRID_ECUDA, GGRID_ENCCL, GGRID_EOVERFLOW = 0, -1, -2, -3, -4, -5
PAD = 0xFFFFFFFF
KERNEL_KINDS = ["ingest_classify", "ingest_alloc", "ingest_scatter", "seed", "flush", "expand",
                "expand_big", "other"]
EXPORTS = ["ggrid_build", "ggrid_ingest", "ggrid_ingest_stage", "ggrid_ingest_commit", "ggrid_query_stage", "ggrid_knn_commit", "ggrid_knn", "ggrid_free", "ggrid_strerror", "ggrid_sync", "ggrid_set_profile", "ggrid_flush_all",
           "ggrid_cell_objects", "ggrid_stats", "ggrid_stats_reset", "ggrid_vertex_cell", "ggrid_zvalue",
           "ggrid_version", "ggrid_shard", "ggrid_query_owner", "ggrid_knn_ex", "ggrid_merge_topk",
           "ggrid_prior_art_clean", "ggrid_prior_art_bundle", "ggrid_wait_stream", "ggrid_signal_stream",
           "ggrid_nccl_unique_id", "ggrid_prior_art_knn"]


class GGridError(RuntimeError):
    def __init__(self, rc: int, what: str):
        self.rc = rc
        super().__init__(f"{what}: {strerror(rc)} ({rc})")


class ggrid_graph(ctypes.Structure):
    _fields_ = [("n_vertices", ctypes.c_uint32), ("n_arcs", ctypes.c_uint32),
                ("src", ctypes.c_void_p), ("dst", ctypes.c_void_p), ("w", ctypes.c_void_p),
                ("x", ctypes.c_void_p), ("y", ctypes.c_void_p)]


ALLTOALL_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.POINTER(ctypes.c_void_p),
                               ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_void_p),
                               ctypes.POINTER(ctypes.c_uint64), ctypes.c_uint32, ctypes.c_void_p)
GGRID_EXCHANGE_AUTO, GGRID_EXCHANGE_LOOPBACK, GGRID_EXCHANGE_NCCL = 0, 1, 2


class ggrid_opts(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("max_k", ctypes.c_uint32), ("max_objects", ctypes.c_uint32),
                ("log_capacity", ctypes.c_uint64), ("delta", ctypes.c_uint32),
                ("seed_neighbors", ctypes.c_uint32), ("profile", ctypes.c_uint32),
                ("t_delta", ctypes.c_uint32), ("stream", ctypes.c_void_p), ("async_ingest", ctypes.c_uint32),
                ("ingest_kernels", ctypes.c_uint32), ("n_gpus", ctypes.c_uint32),
                ("devices", ctypes.POINTER(ctypes.c_int)), ("exchange_kind", ctypes.c_uint32),
                ("n_ranks", ctypes.c_uint32), ("rank", ctypes.c_uint32), ("nccl_id", ctypes.c_void_p),
                ("exchange", ALLTOALL_FN), ("exchange_ctx", ctypes.c_void_p)]


NK = 8


class ggrid_stats_t(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in
                ["n_updates", "n_queries", "knn_calls", "knn_rounds", "cells_flushed", "records_flushed",
                 "objects_written", "arena_used", "arena_capacity", "gc_runs", "launches", "expand_iterations",
                 "expand_vertices", "expand_arcs", "expand_harvested", "expand_objects"]] + [
        ("kernel_launches", ctypes.c_uint64 * NK), ("kernel_ms", ctypes.c_double * NK)] + [
        (n, ctypes.c_uint32) for n in ["n_cells", "cell_size", "delta", "n_vertices", "n_arcs", "max_objects",
                                       "t_delta", "t_now"]] + [("records_expired", ctypes.c_uint64),
                                       ("expand_promotions", ctypes.c_uint64), ("expand_retries", ctypes.c_uint64),
                                       ("seq_rebases", ctypes.c_uint64), ("n_shards", ctypes.c_uint32),
                                       ("exchange_kind", ctypes.c_uint32), ("remote_requests", ctypes.c_uint64),
                                       ("expand_resumes", ctypes.c_uint64)]


class ggrid_prior_art_knn_result(ctypes.Structure):
    _fields_ = [(n, ctypes.c_double) for n in ["ms_clean", "ms_host_index", "ms_gpu", "ms_d2h", "ms_cpu_refine"]] + [
        (n, ctypes.c_uint64) for n in ["cells", "vertices", "bf_iterations", "unresolved", "refine_settled"]] + [
        ("threads", ctypes.c_uint32), ("pad_", ctypes.c_uint32)]


class ggrid_prior_art_result(ctypes.Structure):
    _fields_ = [(n, ctypes.c_double) for n in ["ms_prepare", "ms_shuffle", "ms_collect"]] + [
        (n, ctypes.c_uint64) for n in ["n_buckets", "n_bundles", "table_bytes", "objects_found", "objects_wrong"]]


_lib = None


def lib():
    """Load libggrid.so (raises if it has not been built — no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: run `python -m paper_conf_icde_li0qhdy18_b200.build`")
        L = ctypes.CDLL(LIB_PATH)
        P, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
        sig = {
            "ggrid_build": ([ctypes.POINTER(ggrid_graph), u32, ctypes.POINTER(ggrid_opts), ctypes.POINTER(P)], i32),
            "ggrid_ingest": ([P, P, u64], i32),
            "ggrid_ingest_stage": ([P, P, u64], i32),
            "ggrid_ingest_commit": ([P], i32),
            "ggrid_query_stage": ([P, P, u32], i32),
            "ggrid_knn_commit": ([P, u32, P, P, P], i32),
            "ggrid_knn": ([P, P, u32, u32, P, P], i32),
            "ggrid_free": ([P], i32),
            "ggrid_strerror": ([i32], ctypes.c_char_p),
            "ggrid_flush_all": ([P], i32),
            "ggrid_sync": ([P], i32),
            "ggrid_set_profile": ([P, u32], i32),
            "ggrid_cell_objects": ([P, u32, P, P, P, u32, ctypes.POINTER(u32)], i32),
            "ggrid_stats": ([P, ctypes.POINTER(ggrid_stats_t)], i32),
            "ggrid_stats_reset": ([P], i32),
            "ggrid_vertex_cell": ([P, P], i32),
            "ggrid_zvalue": ([u32, u32], u64),
            "ggrid_version": ([], ctypes.c_char_p),
            "ggrid_shard": ([P, u32, u32], i32),
            "ggrid_query_owner": ([P, P, u32, P], i32),
            "ggrid_knn_ex": ([P, P, u32, u32, P, P, P, P], i32),
            "ggrid_merge_topk": ([P, u32, u32, u32, P, P, P, P], i32),
            "ggrid_prior_art_clean": ([P, u32, u32, u32, P, P, ctypes.POINTER(ggrid_prior_art_result)], i32),
            "ggrid_prior_art_bundle": ([P, P, u32, P, P], i32),
            "ggrid_wait_stream": ([P, P], i32),
            "ggrid_signal_stream": ([P, P], i32),
            "ggrid_nccl_unique_id": ([P], i32),
            "ggrid_prior_art_knn": ([P, P, u32, u32, u32, u32, P, P, ctypes.POINTER(ggrid_prior_art_knn_result)], i32),
        }
        for name, (args, res) in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = res
        _lib = L
    return _lib


def strerror(rc: int) -> str:
    return lib().ggrid_strerror(int(rc)).decode()


def _check(rc: int, what: str):
    if rc != GGRID_OK:
        raise GGridError(rc, what)


def _ptr(a):
    """Raw pointer of a contiguous numpy array or torch tensor (host or device)."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        assert a.flags["C_CONTIGUOUS"]
        return a.ctypes.data
    assert a.is_contiguous()
    return a.data_ptr()


def _u32(a):
    if isinstance(a, np.ndarray):
        return np.ascontiguousarray(a, dtype=np.uint32)
    import torch
    assert a.dtype in (torch.int32, torch.uint32), a.dtype
    return a.contiguous()


def _cuda_stream_of(*arrays):
    """cudaStream_t of torch's current stream on the device of the first CUDA tensor among
    `arrays` (None if there is none): the stream whose queued work produced / consumes them."""
    for a in arrays:
        if a is not None and not isinstance(a, np.ndarray) and getattr(a, "is_cuda", False):
            import torch
            return torch.cuda.current_stream(a.device).cuda_stream
    return None


def _order_inputs(h, *arrays):
    """ggrid_wait_stream on torch's current stream when a CUDA tensor is passed: the library's
    stream then starts after the kernels that produced the tensors (stream 0 is the legacy
    default stream; the C ABI orders after it by itself unless opts.stream was given)."""
    st = _cuda_stream_of(*arrays)
    if st is not None:
        _check(lib().ggrid_wait_stream(h, st), "ggrid_wait_stream")
    return st


# ------------------------------------------------------------------------ the C ABI names
_KEEP = {}  # ctypes objects (callbacks, device lists, ids) that must outlive their handle


def ggrid_build(graph: dict, cell_size: int, *, device: int = 0, max_k: int = 256,
                max_objects: int = 1 << 24, log_capacity: int = 0, delta: int = 0,
                seed_neighbors: bool = True, profile: bool = False, t_delta: int = 0, stream=None,
                async_ingest: bool = False, ingest_kernels: int = 0, n_gpus: int = 0, devices=None,
                exchange_kind: int = 0, n_ranks: int = 0, rank: int = 0, nccl_id: bytes | None = None,
                exchange=None):
    """ggrid_build(graph, cell_size) -> handle (c_void_p).  graph: dict(n_vertices, src, dst, w[, x, y]).

    Multi-GPU (ggrid.h "multi-GPU"): n_gpus/devices (one process, several shards; a repeated
    device = loopback test mode), or n_ranks/rank with nccl_id (128 bytes,
    ggrid_nccl_unique_id) or exchange (a Python all-to-all, see alltoall_callback)."""
    src, dst, w = (np.ascontiguousarray(graph[k], np.uint32) for k in ("src", "dst", "w"))
    x = graph.get("x")
    y = graph.get("y")
    x = None if x is None else np.ascontiguousarray(x, np.int32)
    y = None if y is None else np.ascontiguousarray(y, np.int32)
    g = ggrid_graph(int(graph["n_vertices"]), len(src), src.ctypes.data, dst.ctypes.data, w.ctypes.data,
                    None if x is None else x.ctypes.data, None if y is None else y.ctypes.data)
    keep = []
    dev_arr = None
    if devices is not None:
        dev_arr = (ctypes.c_int * len(devices))(*[int(d) for d in devices])
        keep.append(dev_arr)
        n_gpus = n_gpus or len(devices)
    idbuf = None
    if nccl_id is not None:
        idbuf = ctypes.create_string_buffer(bytes(nccl_id), 128)
        keep.append(idbuf)
    cb = ALLTOALL_FN(0)
    if exchange is not None:
        cb = exchange if isinstance(exchange, ALLTOALL_FN) else ALLTOALL_FN(exchange)
        keep.append(cb)
    o = ggrid_opts(int(device), int(max_k), int(max_objects), int(log_capacity), int(delta),
                   0 if seed_neighbors else 2, int(profile), int(t_delta), stream,
                   1 if async_ingest else 0, int(ingest_kernels), int(n_gpus),
                   ctypes.cast(dev_arr, ctypes.POINTER(ctypes.c_int)) if dev_arr is not None else None,
                   int(exchange_kind), int(n_ranks), int(rank),
                   ctypes.cast(idbuf, ctypes.c_void_p) if idbuf is not None else None, cb, None)
    h = ctypes.c_void_p()
    _check(lib().ggrid_build(ctypes.byref(g), int(cell_size), ctypes.byref(o), ctypes.byref(h)), "ggrid_build")
    if keep:
        _KEEP[h.value] = keep
    return h


def ggrid_nccl_unique_id() -> bytes:
    """A fresh 128-byte ncclUniqueId for ggrid_build(n_ranks=..., nccl_id=...)."""
    buf = ctypes.create_string_buffer(128)
    _check(lib().ggrid_nccl_unique_id(buf), "ggrid_nccl_unique_id")
    return buf.raw


def alltoall_callback(torch_group=None):
    """An opts.exchange all-to-all over torch.distributed (any backend; gloo exchanges through
    host memory).  Device segments are viewed as uint8 CUDA tensors of this rank's device."""
    import torch
    import torch.distributed as dist

    def fn(ctx, send, sbytes, recv, rbytes, n_ranks, stream):
        try:
            dev = torch.cuda.current_device()
            ins, outs = [], []
            for p in range(n_ranks):
                ins.append(_u8_view(send[p], sbytes[p], dev))
                outs.append(_u8_view(recv[p], rbytes[p], dev))
            ssz = [int(sbytes[p]) for p in range(n_ranks)]
            rsz = [int(rbytes[p]) for p in range(n_ranks)]
            host = dist.get_backend(torch_group) == "gloo"  # (gloo: CPU tensors, no list all_to_all)
            cat_in = torch.cat(ins) if sum(ssz) else torch.empty(0, dtype=torch.uint8, device=f"cuda:{dev}")
            cat_in = cat_in.cpu() if host else cat_in
            cat_out = torch.empty(sum(rsz), dtype=torch.uint8, device="cpu" if host else f"cuda:{dev}")
            dist.all_to_all_single(cat_out, cat_in, rsz, ssz, group=torch_group)
            off = 0
            for p in range(n_ranks):
                if rsz[p]:
                    outs[p].copy_(cat_out[off:off + rsz[p]])
                off += rsz[p]
            torch.cuda.synchronize(dev)
            return 0
        except Exception as e:  # (reported to the library as a failed exchange: ENCCL)
            import sys
            print("ggrid exchange callback failed:", repr(e), file=sys.stderr)
            return 1

    return ALLTOALL_FN(fn)


def _u8_view(ptr, nbytes, dev):
    """A uint8 CUDA tensor over nbytes of device memory at ptr (no copy)."""
    import torch

    n = int(nbytes)
    if n == 0 or not ptr:
        return torch.empty(0, dtype=torch.uint8, device=f"cuda:{dev}")

    class _Arr:
        __cuda_array_interface__ = {"shape": (n,), "typestr": "|u1", "data": (int(ptr), False), "version": 3}

    return torch.as_tensor(_Arr(), device=f"cuda:{dev}")


def ggrid_ingest(h, updates, n: int | None = None):
    """Append updates: (n, 4) u32 (obj, edge, offset, t) numpy array or torch tensor."""
    u = _u32(updates)
    cnt = int(u.shape[0]) if n is None else int(n)
    st = _order_inputs(h, u)
    _check(lib().ggrid_ingest(h, _ptr(u), cnt), "ggrid_ingest")
    if st is not None:  # (async ingest) the caller's later work on u waits for the kernels reading it
        _check(lib().ggrid_signal_stream(h, st), "ggrid_signal_stream")


def ggrid_sync(h):
    """Drain the stream; raises the deferred error of a rejected asynchronous ingest batch."""
    _check(lib().ggrid_sync(h), "ggrid_sync")


def ggrid_set_profile(h, mask: int):
    """Kinds of launches timed with CUDA events: bit 0 = all, bit k+1 = kind k (K_*)."""
    _check(lib().ggrid_set_profile(h, int(mask)), "ggrid_set_profile")


def ggrid_ingest_stage(h, updates):
    """Start the asynchronous copy of a batch (keep `updates` alive until the commit)."""
    u = _u32(updates)
    _order_inputs(h, u)
    _check(lib().ggrid_ingest_stage(h, _ptr(u), int(u.shape[0])), "ggrid_ingest_stage")
    return u


def ggrid_ingest_commit(h):
    _check(lib().ggrid_ingest_commit(h), "ggrid_ingest_commit")


def ggrid_query_stage(h, queries):
    """Start the asynchronous copy of a query batch (keep `queries` alive until knn_commit)."""
    q = _u32(queries)
    _order_inputs(h, q)
    _check(lib().ggrid_query_stage(h, _ptr(q), int(q.shape[0])), "ggrid_query_stage")
    return q


def ggrid_knn_commit(h, k: int, out_obj, out_dist):
    """Answer the oldest staged query batch into out_obj / out_dist (preallocated, (n, k))."""
    n = ctypes.c_uint32(0)
    _order_inputs(h, out_obj, out_dist)
    _check(lib().ggrid_knn_commit(h, int(k), _ptr(out_obj), _ptr(out_dist), ctypes.byref(n)),
           "ggrid_knn_commit")
    return out_obj, out_dist


def ggrid_knn(h, queries, k: int, out_obj=None, out_dist=None):
    """Answer queries ((n, 2) u32 (edge, offset)); returns (out_obj, out_dist) of shape (n, k).

    Outputs default to numpy arrays; pass preallocated torch tensors (int32/uint32, host or
    CUDA) to receive them in place."""
    q = _u32(queries)
    nq = int(q.shape[0])
    if out_obj is None:
        out_obj = np.empty((nq, k), np.uint32)
    if out_dist is None:
        out_dist = np.empty((nq, k), np.uint32)
    _order_inputs(h, q, out_obj, out_dist)
    _check(lib().ggrid_knn(h, _ptr(q), nq, int(k), _ptr(out_obj), _ptr(out_dist)), "ggrid_knn")
    return out_obj, out_dist


def ggrid_knn_ex(h, queries, k: int, bound=None, out_obj=None, out_dist=None, out_remote=None):
    """ggrid_knn with an optional per-query distance bound (n,) u32 and per-query remote-rank
    masks (n,) u64 (pass an array/tensor, or True for a new numpy array).  Returns
    (out_obj, out_dist, out_remote)."""
    q = _u32(queries)
    nq = int(q.shape[0])
    if out_obj is None:
        out_obj = np.empty((nq, k), np.uint32)
    if out_dist is None:
        out_dist = np.empty((nq, k), np.uint32)
    if out_remote is True:
        out_remote = np.empty(nq, np.uint64)
    b = None if bound is None else _u32(bound)
    _order_inputs(h, q, b, out_obj, out_dist, None if out_remote is None or out_remote is True else out_remote)
    _check(lib().ggrid_knn_ex(h, _ptr(q), nq, int(k), _ptr(b), _ptr(out_obj), _ptr(out_dist), _ptr(out_remote)),
           "ggrid_knn_ex")
    return out_obj, out_dist, out_remote


def ggrid_shard(h, n_ranks: int, rank: int):
    _check(lib().ggrid_shard(h, int(n_ranks), int(rank)), "ggrid_shard")


def ggrid_query_owner(h, queries, out_rank=None):
    q = _u32(queries)
    nq = int(q.shape[0])
    if out_rank is None:
        out_rank = np.empty(nq, np.uint32)
    _order_inputs(h, q, out_rank)
    _check(lib().ggrid_query_owner(h, _ptr(q), nq, _ptr(out_rank)), "ggrid_query_owner")
    return out_rank


def ggrid_merge_topk(h, lists_obj, lists_dist, out_obj=None, out_dist=None):
    """lists_obj / lists_dist: (n_lists, n_q, k) u32; returns (out_obj, out_dist) (n_q, k)."""
    lo, ld = _u32(lists_obj), _u32(lists_dist)
    L, nq, k = (int(x) for x in lo.shape)
    if out_obj is None:
        out_obj = np.empty((nq, k), np.uint32)
    if out_dist is None:
        out_dist = np.empty((nq, k), np.uint32)
    _order_inputs(h, lo, ld, out_obj, out_dist)
    _check(lib().ggrid_merge_topk(h, L, nq, k, _ptr(lo), _ptr(ld), _ptr(out_obj), _ptr(out_dist)),
           "ggrid_merge_topk")
    return out_obj, out_dist


def ggrid_prior_art_clean(h, eta: int = 5, bucket_size: int = 128, write_mode: int = 0,
                          max_objects: int | None = None):
    """The paper's message cleaning (Alg. 2-3 + GPU_Collect) as a read-only comparison pass.
    Returns (result dict, edge, off) — edge/off per object (PAD: none) if max_objects given."""
    r = ggrid_prior_art_result()
    e = o = None
    if max_objects:
        e = np.empty(max_objects, np.uint32)
        o = np.empty(max_objects, np.uint32)
    _check(lib().ggrid_prior_art_clean(h, int(eta), int(bucket_size), int(write_mode), _ptr(e), _ptr(o),
                                       ctypes.byref(r)), "ggrid_prior_art_clean")
    return {f: getattr(r, f) for f, _ in ggrid_prior_art_result._fields_}, e, o


def ggrid_prior_art_knn(h, queries, k: int, rho: float = 1.8, threads: int = 0):
    """The paper's query pipeline (Alg. 4-6: GPU candidates, CPU-thread Refine_kNN) as a
    comparison path.  Returns (obj, dist, result dict); answers have ggrid_knn's format."""
    q = _u32(queries)
    nq = int(q.shape[0])
    oo = np.empty((nq, k), np.uint32)
    od = np.empty((nq, k), np.uint32)
    r = ggrid_prior_art_knn_result()
    _order_inputs(h, q)
    _check(lib().ggrid_prior_art_knn(h, _ptr(q), nq, int(k), int(round(rho * 100)), int(threads), _ptr(oo), _ptr(od),
                                     ctypes.byref(r)), "ggrid_prior_art_knn")
    return oo, od, {f: getattr(r, f) for f, _ in ggrid_prior_art_knn_result._fields_ if f != "pad_"}


def ggrid_prior_art_bundle(obj, key, eta: int):
    """Alg. 3 Step 1 (cache-and-shuffle) on one bundle; returns (obj, key) per lane after it."""
    ob = np.ascontiguousarray(obj, np.uint32)
    ky = np.ascontiguousarray(key, np.uint64)
    oo = np.empty_like(ob)
    ok = np.empty_like(ky)
    _check(lib().ggrid_prior_art_bundle(_ptr(ob), _ptr(ky), int(eta), _ptr(oo), _ptr(ok)), "ggrid_prior_art_bundle")
    return oo, ok


def ggrid_wait_stream(h, stream=None):
    """Later calls on h start after the work queued on `stream` (torch.cuda.Stream, raw
    cudaStream_t int, or None = torch's current stream)."""
    _check(lib().ggrid_wait_stream(h, _stream_handle(stream)), "ggrid_wait_stream")


def ggrid_signal_stream(h, stream=None):
    """Work queued on `stream` from now on starts after everything h has queued so far."""
    _check(lib().ggrid_signal_stream(h, _stream_handle(stream)), "ggrid_signal_stream")


def _stream_handle(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    return int(getattr(stream, "cuda_stream", stream))


def ggrid_free(h):
    if h:
        lib().ggrid_free(h)
        _KEEP.pop(h.value if hasattr(h, "value") else h, None)


def ggrid_flush_all(h):
    _check(lib().ggrid_flush_all(h), "ggrid_flush_all")


def ggrid_cell_objects(h, cell: int, cap: int = 1 << 16):
    obj = np.empty(cap, np.uint32)
    edge = np.empty(cap, np.uint32)
    off = np.empty(cap, np.uint32)
    n = ctypes.c_uint32()
    _check(lib().ggrid_cell_objects(h, int(cell), obj.ctypes.data, edge.ctypes.data, off.ctypes.data, cap,
                                    ctypes.byref(n)), "ggrid_cell_objects")
    if n.value > cap:
        return ggrid_cell_objects(h, cell, int(n.value))
    m = n.value
    return obj[:m].copy(), edge[:m].copy(), off[:m].copy()


def ggrid_stats(h) -> dict:
    s = ggrid_stats_t()
    _check(lib().ggrid_stats(h, ctypes.byref(s)), "ggrid_stats")
    d = {f: getattr(s, f) for f, _ in ggrid_stats_t._fields_ if f not in ("kernel_launches", "kernel_ms")}
    d["kernel_launches"] = dict(zip(KERNEL_KINDS, list(s.kernel_launches)))
    d["kernel_ms"] = dict(zip(KERNEL_KINDS, list(s.kernel_ms)))
    return d


def ggrid_stats_reset(h):
    _check(lib().ggrid_stats_reset(h), "ggrid_stats_reset")


def ggrid_vertex_cell(h, n_vertices: int):
    out = np.empty(n_vertices, np.uint32)
    _check(lib().ggrid_vertex_cell(h, out.ctypes.data), "ggrid_vertex_cell")
    return out


def ggrid_zvalue(x: int, y: int) -> int:
    return int(lib().ggrid_zvalue(int(x), int(y)))


def ggrid_version() -> str:
    return lib().ggrid_version().decode()


class GGrid:
    """Owning wrapper: GGrid(graph, cell_size, **opts).ingest(u).knn(q, k)."""

    def __init__(self, graph: dict, cell_size: int, **opts):
        self.n_vertices = int(graph["n_vertices"])
        self._staged = []
        self._qstaged = []
        self.h = ggrid_build(graph, cell_size, **opts)

    def ingest(self, updates):
        ggrid_ingest(self.h, updates)
        return self

    def wait_stream(self, stream=None):
        ggrid_wait_stream(self.h, stream)
        return self

    def signal_stream(self, stream=None):
        ggrid_signal_stream(self.h, stream)
        return self

    def sync(self):
        ggrid_sync(self.h)
        return self

    def set_profile(self, mask: int):
        ggrid_set_profile(self.h, mask)
        return self

    def ingest_stage(self, updates):
        """Pipelined ingest: copy now, ingest at ingest_commit (P@45017-45625)."""
        self._staged.append(ggrid_ingest_stage(self.h, updates))
        return self

    def ingest_commit(self):
        ggrid_ingest_commit(self.h)
        self._staged.pop(0)
        return self

    def knn(self, queries, k: int, out_obj=None, out_dist=None):
        return ggrid_knn(self.h, queries, k, out_obj, out_dist)

    def query_stage(self, queries):
        """Pipelined queries: copy now, answer at knn_commit."""
        self._qstaged.append(ggrid_query_stage(self.h, queries))
        return self

    def knn_commit(self, k: int, out_obj, out_dist):
        r = ggrid_knn_commit(self.h, k, out_obj, out_dist)
        self._qstaged.pop(0)
        return r

    def knn_ex(self, queries, k: int, bound=None, out_obj=None, out_dist=None, out_remote=None):
        return ggrid_knn_ex(self.h, queries, k, bound, out_obj, out_dist, out_remote)

    def shard(self, n_ranks: int, rank: int):
        ggrid_shard(self.h, n_ranks, rank)
        return self

    def query_owner(self, queries, out_rank=None):
        return ggrid_query_owner(self.h, queries, out_rank)

    def merge_topk(self, lists_obj, lists_dist, out_obj=None, out_dist=None):
        return ggrid_merge_topk(self.h, lists_obj, lists_dist, out_obj, out_dist)

    def prior_art_clean(self, eta: int = 5, bucket_size: int = 128, write_mode: int = 0, locations: bool = False):
        return ggrid_prior_art_clean(self.h, eta, bucket_size, write_mode,
                                     self.stats()["max_objects"] if locations else None)

    def prior_art_knn(self, queries, k: int, rho: float = 1.8, threads: int = 0):
        return ggrid_prior_art_knn(self.h, queries, k, rho, threads)

    def flush_all(self):
        ggrid_flush_all(self.h)

    def cell_objects(self, cell: int):
        return ggrid_cell_objects(self.h, cell)

    def vertex_cell(self):
        return ggrid_vertex_cell(self.h, self.n_vertices)

    def stats(self):
        return ggrid_stats(self.h)

    def stats_reset(self):
        ggrid_stats_reset(self.h)

    def close(self):
        if self.h:
            ggrid_free(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
