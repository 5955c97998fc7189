"""Seeded synthetic graph generators (input infrastructure).

The paper's workloads are real SNAP/LAW/KONECT graphs (Table I,
P:L400-423), unavailable offline; BASELINE.json's configs are synthetic graphs
of the same shape.  This module (ctypes over ``kcgen/libkcgen.so``) produces
them deterministically from ``(kind, params, seed)`` on the host (small graphs,
CPU tests) or on the device (full-size configs), byte-identically.  It holds
no k-core arithmetic: both the CUDA path and the CPU oracle consume its CSRs.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, replace

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "libkcgen.so")
_lib = None

RMAT, ER, CHUNGLU = 1, 2, 3


class _Params(ctypes.Structure):
    _fields_ = [
        ("kind", ctypes.c_int32), ("scale", ctypes.c_int32), ("n", ctypes.c_int64),
        ("num_edges", ctypes.c_int64), ("a", ctypes.c_double), ("b", ctypes.c_double),
        ("c", ctypes.c_double), ("gamma", ctypes.c_double), ("seed", ctypes.c_uint64),
        ("permute", ctypes.c_int32), ("reserved", ctypes.c_int32),
    ]


@dataclass(frozen=True)
class GraphSpec:
    kind: int
    scale: int = 0
    n: int = 0
    num_edges: int = 0
    a: float = 0.57
    b: float = 0.19
    c: float = 0.19
    gamma: float = 2.1
    seed: int = 1
    permute: int = 1
    name: str = ""

    @property
    def num_vertices(self) -> int:
        return (1 << self.scale) if self.kind == RMAT else self.n

    def with_seed(self, seed: int) -> "GraphSpec":
        return replace(self, seed=seed)

    def _c(self) -> _Params:
        return _Params(self.kind, self.scale, self.n, self.num_edges, self.a, self.b, self.c,
                       self.gamma, self.seed, self.permute, 0)


def rmat(scale: int, edge_factor: int, seed: int = 1, a=0.57, b=0.19, c=0.19) -> GraphSpec:
    """Graph500-style R-MAT: (edge_factor * 2^scale) draws, hashed vertex ids."""
    return GraphSpec(RMAT, scale=scale, num_edges=edge_factor << scale, a=a, b=b, c=c, seed=seed,
                     name=f"rmat-s{scale}-ef{edge_factor}")


def er(n: int, avg_deg: int, seed: int = 1) -> GraphSpec:
    """Erdos-Renyi G(n, M) with M = n*avg_deg/2 uniform pairs."""
    return GraphSpec(ER, n=n, num_edges=n * avg_deg // 2, seed=seed, permute=0,
                     name=f"er-n{n}-d{avg_deg}")


def chunglu(n: int, gamma: float, draws: int, seed: int = 1) -> GraphSpec:
    """Chung-Lu power law: w_i = (i+1)^(-1/(gamma-1)), `draws` i.i.d. endpoint pairs."""
    return GraphSpec(CHUNGLU, n=n, num_edges=draws, gamma=gamma, seed=seed,
                     name=f"chunglu-n{n}-g{gamma}-M{draws}")


# BASELINE.json configs; "4M" = 2^22 (reading R9).
CHUNGLU_C3_DRAWS = 86_800_000
CONFIGS = {
    "C1": rmat(16, 16),
    "C2": er(1 << 22, 32),
    "C3": chunglu(1 << 22, 2.1, CHUNGLU_C3_DRAWS),
    "C4": rmat(24, 32),
    "C5": rmat(27, 32),
}


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB):
            raise RuntimeError(f"{_LIB} missing: run `make` (or __graft_entry__.build())")
        lib = ctypes.CDLL(_LIB)
        P = ctypes.POINTER(_Params)
        lib.kcg_num_vertices.argtypes = [P]
        lib.kcg_num_vertices.restype = ctypes.c_int64
        lib.kcg_build_cdf.argtypes = [P, ctypes.POINTER(ctypes.c_double)]
        lib.kcg_edge.argtypes = [P, ctypes.POINTER(ctypes.c_double), ctypes.c_int64,
                                 ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64)]
        lib.kcg_host_generate.argtypes = [P, ctypes.c_int64, ctypes.c_int64,
                                          ctypes.POINTER(ctypes.c_int64),
                                          ctypes.POINTER(ctypes.c_int32), ctypes.c_int64]
        lib.kcg_host_generate.restype = ctypes.c_int64
        lib.kcg_device_generate.argtypes = [P, ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p,
                                            ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p]
        lib.kcg_device_generate.restype = ctypes.c_int64
        _lib = lib
    return _lib


def edge(spec: GraphSpec, i: int, cdf=None):
    u = ctypes.c_int64()
    v = ctypes.c_int64()
    cp = None
    if spec.kind == CHUNGLU:
        cdf = build_cdf(spec) if cdf is None else cdf
        cp = cdf.ctypes.data_as(ctypes.POINTER(ctypes.c_double))
    p = spec._c()
    rc = _load().kcg_edge(ctypes.byref(p), cp, i, ctypes.byref(u), ctypes.byref(v))
    if rc != 0:
        raise ValueError(f"kcg_edge: {rc}")
    return u.value, v.value


def build_cdf(spec: GraphSpec) -> np.ndarray:
    cdf = np.empty(spec.n, dtype=np.float64)
    p = spec._c()
    if _load().kcg_build_cdf(ctypes.byref(p), cdf.ctypes.data_as(ctypes.POINTER(ctypes.c_double))):
        raise ValueError("kcg_build_cdf failed")
    return cdf


def generate_host(spec: GraphSpec, v_begin: int = 0, v_end: int | None = None):
    """(rowptr int64[nl+1], colidx int32[arcs]) on the host."""
    n = spec.num_vertices
    v_end = n if v_end is None else v_end
    p = spec._c()
    rowptr = np.empty(v_end - v_begin + 1, dtype=np.int64)
    cap = 2 * spec.num_edges
    colidx = np.empty(max(cap, 1), dtype=np.int32)
    m = _load().kcg_host_generate(ctypes.byref(p), v_begin, v_end,
                                  rowptr.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                  colidx.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)), cap)
    if m < 0:
        raise RuntimeError(f"kcg_host_generate failed: {m}")
    return rowptr, colidx[:m].copy()


def generate_device(spec: GraphSpec, v_begin: int = 0, v_end: int | None = None, device=None):
    """(rowptr, colidx) as torch CUDA tensors, generated on the device."""
    import torch

    device = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
    n = spec.num_vertices
    v_end = n if v_end is None else v_end
    p = spec._c()
    lib = _load()
    with torch.cuda.device(device):
        stream = torch.cuda.current_stream(device).cuda_stream
        full = (v_begin == 0 and v_end == n)
        cap = 2 * spec.num_edges if full else lib.kcg_device_generate(
            ctypes.byref(p), v_begin, v_end, None, None, 0, stream)
        if cap < 0:
            raise RuntimeError(f"kcg_device_generate(count) failed: {cap}")
        rowptr = torch.empty(v_end - v_begin + 1, dtype=torch.int64, device=device)
        colidx = torch.empty(max(cap, 1), dtype=torch.int32, device=device)
        m = lib.kcg_device_generate(ctypes.byref(p), v_begin, v_end, rowptr.data_ptr(),
                                    colidx.data_ptr(), cap, stream)
        if m < 0:
            raise RuntimeError(f"kcg_device_generate failed: {m}")
        return rowptr, colidx[:m]


def generate_device_chunked(spec: GraphSpec, chunks: int = 16, device=None):
    """The whole graph's CSR on the device, generated in `chunks` owner ranges
    (each range regenerates every edge and keeps the arcs whose source it
    owns), written straight into one colidx buffer of capacity 2*num_edges.
    For graphs whose one-shot sort buffers would not fit next to the CSR
    (C5: 8.6 G candidate arcs).  Byte-identical to generate_device(spec)."""
    import torch

    device = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
    n = spec.num_vertices
    p = spec._c()
    lib = _load()
    with torch.cuda.device(device):
        stream = torch.cuda.current_stream(device).cuda_stream
        cap = 2 * spec.num_edges
        colidx = torch.empty(cap, dtype=torch.int32, device=device)
        rowptr = torch.empty(n + 1, dtype=torch.int64, device=device)
        rowptr[0] = 0
        off = 0
        bounds = [n * i // chunks for i in range(chunks + 1)]
        for vb, ve in zip(bounds[:-1], bounds[1:]):
            rp = torch.empty(ve - vb + 1, dtype=torch.int64, device=device)
            m = lib.kcg_device_generate(ctypes.byref(p), vb, ve, rp.data_ptr(), colidx.data_ptr() + 4 * off,
                                        cap - off, stream)
            if m < 0:
                raise RuntimeError(f"kcg_device_generate({vb},{ve}) failed: {m}")
            rowptr[vb + 1:ve + 1] = rp[1:] + off
            off += m
            del rp
        torch.cuda.synchronize(device)
        return rowptr, colidx[:off]


def csr_from_edges(n: int, edges):
    """CSR of a hand-written edge list: symmetrised, self-loops dropped,
    duplicates merged, rows sorted (reading R2)."""
    adj = [set() for _ in range(n)]
    for u, v in edges:
        if u == v:
            continue
        adj[u].add(v)
        adj[v].add(u)
    rowptr = np.zeros(n + 1, dtype=np.int64)
    for v in range(n):
        rowptr[v + 1] = rowptr[v] + len(adj[v])
    colidx = np.fromiter((u for v in range(n) for u in sorted(adj[v])), dtype=np.int32,
                         count=int(rowptr[n]))
    return rowptr, colidx


def disjoint_union(graphs):
    """Concatenate CSRs (relabelling ids) into one graph."""
    rps, cis, off, aoff = [], [], 0, 0
    for rp, ci in graphs:
        rp = np.asarray(rp, dtype=np.int64)
        ci = np.asarray(ci, dtype=np.int32)
        rps.append(rp[:-1] + aoff)
        cis.append(ci + off)
        off += rp.shape[0] - 1
        aoff += int(rp[-1])
    rowptr = np.concatenate(rps + [np.array([aoff], dtype=np.int64)])
    colidx = np.concatenate(cis) if cis else np.zeros(0, dtype=np.int32)
    return rowptr, colidx.astype(np.int32)
