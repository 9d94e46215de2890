"""CPU oracle (TEST INFRASTRUCTURE ONLY).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / `--impl reference`
legs may import this package.  The product package never imports it and shares no
code with it; see oracle/oracle.cpp for what is computed and which PAPER.md passages
each step follows.

The Python side is argument marshalling over ctypes plus two convenience helpers that
are themselves plain definitions (`snapshot_objects`: the objects that exist with their
latest location).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")
PAD = 0xFFFFFFFF
FULL, EARLY = 0, 1


def build(force: bool = False) -> str:
    """Compile oracle.cpp -> liboracle.so with g++ (plain -O2, no tuning)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-pthread",
                               "-o", _LIB, _SRC])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        u32, u64, i32 = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
        L.oracle_snapshot.argtypes = [u64, P, u64, u32, P, P, P, P, P]
        L.oracle_snapshot.restype = i32
        L.oracle_vertex_dist.argtypes = [u32, u32, P, P, P, u32, u32, P]
        L.oracle_vertex_dist.restype = i32
        L.oracle_knn.argtypes = [u32, u32, P, P, P, u32, P, P, P, u32, P, P, u32, i32, i32, P, P]
        L.oracle_knn.restype = i32
        L.oracle_hardware_threads.argtypes = []
        L.oracle_hardware_threads.restype = i32
        _lib = L
    return _lib


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def _u32(a):
    return np.ascontiguousarray(a, dtype=np.uint32)


def hardware_threads() -> int:
    return int(lib().oracle_hardware_threads())


class Snapshot:
    """Latest update per object by max (t, seq) (oracle_snapshot; step 1)."""

    def __init__(self, n_obj_cap: int):
        self.cap = int(n_obj_cap)
        self.has = np.zeros(self.cap, np.uint8)
        self.edge = np.zeros(self.cap, np.uint32)
        self.off = np.zeros(self.cap, np.uint32)
        self.t = np.zeros(self.cap, np.uint32)
        self.seq = np.zeros(self.cap, np.uint64)
        self.n_seen = 0

    def apply(self, updates: np.ndarray):
        u = _u32(updates).reshape(-1, 4)
        rc = lib().oracle_snapshot(len(u), _p(u), self.n_seen, self.cap, _p(self.has), _p(self.edge),
                                   _p(self.off), _p(self.t), _p(self.seq))
        if rc != 0:
            raise ValueError("object id out of range")
        self.n_seen += len(u)
        return self

    def objects(self):
        """(ids, edge, offset) of every object that exists, ascending id."""
        ids = np.flatnonzero(self.has).astype(np.uint32)
        return ids, self.edge[ids].copy(), self.off[ids].copy()


def snapshot_objects(updates: np.ndarray, n_obj_cap: int | None = None):
    u = _u32(updates).reshape(-1, 4)
    cap = int(n_obj_cap if n_obj_cap is not None else (int(u[:, 0].max()) + 1 if len(u) else 1))
    return Snapshot(cap).apply(u).objects()


def vertex_dist(graph, q_edge: int, q_off: int) -> np.ndarray:
    """u64 distances from location (q_edge, q_off) to every vertex (2^64-1 = unreachable)."""
    src, dst, w = _u32(graph["src"]), _u32(graph["dst"]), _u32(graph["w"])
    D = np.empty(graph["n_vertices"], np.uint64)
    rc = lib().oracle_vertex_dist(graph["n_vertices"], len(src), _p(src), _p(dst), _p(w),
                                  int(q_edge), int(q_off), _p(D))
    if rc != 0:
        raise ValueError("bad graph or query")
    return D


def knn(graph, obj_ids, obj_edge, obj_off, queries, k: int, mode: int = FULL, threads: int = 0):
    """k nearest (obj, dist) per query, ascending (dist, obj), padded with 0xFFFFFFFF."""
    src, dst, w = _u32(graph["src"]), _u32(graph["dst"]), _u32(graph["w"])
    oi, oe, oo = _u32(obj_ids), _u32(obj_edge), _u32(obj_off)
    q = _u32(queries).reshape(-1, 2)
    qe, qo = np.ascontiguousarray(q[:, 0]), np.ascontiguousarray(q[:, 1])
    nq = len(q)
    out_o = np.empty((nq, k), np.uint32)
    out_d = np.empty((nq, k), np.uint32)
    rc = lib().oracle_knn(graph["n_vertices"], len(src), _p(src), _p(dst), _p(w), len(oi), _p(oi), _p(oe),
                          _p(oo), nq, _p(qe), _p(qo), int(k), int(mode), int(threads), _p(out_o), _p(out_d))
    if rc != 0:
        raise ValueError("bad oracle input")
    return out_o, out_d


def knn_from_updates(graph, updates, queries, k: int, mode: int = FULL, threads: int = 0,
                     n_obj_cap: int | None = None):
    ids, e, o = snapshot_objects(updates, n_obj_cap)
    return knn(graph, ids, e, o, queries, k, mode, threads)
