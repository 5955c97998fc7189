"""CPU oracle for k-core decomposition -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product path (``paper_conf_icde_ahmady0gcz23_b200``) never imports it and
shares no code with it.

Thin ctypes wrapper over ``oracle/kcore_oracle.c`` (plain serial C); see that
file's header for the paper passages each function follows:

* :func:`bz_core`             -- Batagelj-Zaversnik peeling [30].
* :func:`core_by_deletion`    -- the k-core definition by repeated deletion.
* :func:`core_smallest_last`  -- smallest-last min-degree removal (ref [58]).
* :func:`core_subsets`        -- literal subset definition, n <= 20.
* :func:`hindex`              -- MPM h-index operator (Fig. 2).
* :func:`kcore_members`       -- the k-core by its definition (repeated deletion).
* :func:`induced_csr`         -- induced subgraph G[S], renumbered by increasing id.
* :func:`mpm`                 -- synchronous MPM h-index iteration.
* :func:`check_invariants`, :func:`check_certificate`, :func:`validate_csr`.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "kcore_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

I64P = ctypes.POINTER(ctypes.c_int64)
I32P = ctypes.POINTER(ctypes.c_int32)


def build(force: bool = False) -> str:
    """Compile the oracle (plain C, -O2, single thread)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", _SRC, "-o", _LIB])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.oracle_bz_core.argtypes = [ctypes.c_int64, I64P, I32P, I32P, I32P]
        lib.oracle_core_by_deletion.argtypes = [ctypes.c_int64, I64P, I32P, I32P]
        lib.oracle_core_smallest_last.argtypes = [ctypes.c_int64, I64P, I32P, I32P]
        lib.oracle_core_subsets_mask.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_uint32), I32P]
        lib.oracle_core_subsets_mask.restype = None
        lib.oracle_exhaustive_check.argtypes = [ctypes.c_int, I64P]
        lib.oracle_exhaustive_check.restype = ctypes.c_int64
        lib.oracle_hindex.argtypes = [I32P, ctypes.c_int64]
        lib.oracle_hindex.restype = ctypes.c_int32
        lib.oracle_check_invariants.argtypes = [ctypes.c_int64, I64P, I32P, I32P]
        lib.oracle_check_certificate.argtypes = [ctypes.c_int64, I64P, I32P, I32P, I32P]
        lib.oracle_validate_csr.argtypes = [ctypes.c_int64, ctypes.c_int64, I64P, I32P]
        U8P = ctypes.POINTER(ctypes.c_uint8)
        lib.oracle_kcore_members.argtypes = [ctypes.c_int64, I64P, I32P, ctypes.c_int64, U8P]
        lib.oracle_induced_csr.argtypes = [ctypes.c_int64, I64P, I32P, U8P, I64P, I64P, I64P, I32P, I32P]
        lib.oracle_mpm.argtypes = [ctypes.c_int64, I64P, I32P, ctypes.c_int64, I32P, I64P]
        _lib = lib
    return _lib


def _csr(rowptr, colidx):
    rp = np.ascontiguousarray(np.asarray(rowptr), dtype=np.int64)
    ci = np.ascontiguousarray(np.asarray(colidx), dtype=np.int32)
    n = rp.shape[0] - 1
    return rp, ci, n


def _p64(a):
    return a.ctypes.data_as(I64P)


def _p32(a):
    return a.ctypes.data_as(I32P) if a is not None else None


def bz_core(rowptr, colidx, return_order: bool = False):
    """Core numbers by BZ [30]; optionally also its removal (degeneracy) order."""
    rp, ci, n = _csr(rowptr, colidx)
    core = np.empty(n, dtype=np.int32)
    vert = np.empty(n, dtype=np.int32) if return_order else None
    rc = _load().oracle_bz_core(n, _p64(rp), _p32(ci), _p32(core), _p32(vert))
    if rc != 0:
        raise RuntimeError(f"oracle_bz_core failed: {rc}")
    return (core, vert) if return_order else core


def core_by_deletion(rowptr, colidx):
    rp, ci, n = _csr(rowptr, colidx)
    core = np.empty(n, dtype=np.int32)
    if _load().oracle_core_by_deletion(n, _p64(rp), _p32(ci), _p32(core)) != 0:
        raise RuntimeError("oracle_core_by_deletion failed")
    return core


def core_smallest_last(rowptr, colidx):
    rp, ci, n = _csr(rowptr, colidx)
    core = np.empty(n, dtype=np.int32)
    if _load().oracle_core_smallest_last(n, _p64(rp), _p32(ci), _p32(core)) != 0:
        raise RuntimeError("oracle_core_smallest_last failed")
    return core


def core_subsets(rowptr, colidx):
    """Literal definition over all vertex subsets (n <= 20)."""
    rp, ci, n = _csr(rowptr, colidx)
    if n > 20:
        raise ValueError("core_subsets is exponential; n <= 20 only")
    adj = np.zeros(max(n, 1), dtype=np.uint32)
    for v in range(n):
        for e in range(rp[v], rp[v + 1]):
            adj[v] |= np.uint32(1 << int(ci[e]))
    core = np.empty(max(n, 1), dtype=np.int32)
    _load().oracle_core_subsets_mask(n, adj.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)), _p32(core))
    return core[:n]


def exhaustive_check(n: int):
    """(#disagreeing graphs, #graphs) over every labelled graph on n<=7 vertices."""
    cnt = ctypes.c_int64(0)
    bad = _load().oracle_exhaustive_check(n, ctypes.byref(cnt))
    return int(bad), int(cnt.value)


def hindex(values) -> int:
    a = np.ascontiguousarray(np.asarray(values), dtype=np.int32)
    return int(_load().oracle_hindex(_p32(a), a.shape[0]))


def check_invariants(rowptr, colidx, core) -> int:
    """Bitmask of violated invariants (I1=1, I2=2, I3=4, I5=8, I6=16); 0 = ok."""
    rp, ci, n = _csr(rowptr, colidx)
    c = np.ascontiguousarray(np.asarray(core), dtype=np.int32)
    return int(_load().oracle_check_invariants(n, _p64(rp), _p32(ci), _p32(c)))


def check_certificate(rowptr, colidx, core, order) -> int:
    """0 if `order` certifies `core` from above (I4)."""
    rp, ci, n = _csr(rowptr, colidx)
    c = np.ascontiguousarray(np.asarray(core), dtype=np.int32)
    o = np.ascontiguousarray(np.asarray(order), dtype=np.int32)
    return int(_load().oracle_check_certificate(n, _p64(rp), _p32(ci), _p32(c), _p32(o)))


def validate_csr(rowptr, colidx) -> int:
    """0 if the CSR is a valid simple undirected graph (sorted, symmetric)."""
    rp, ci, n = _csr(rowptr, colidx)
    return int(_load().oracle_validate_csr(n, ci.shape[0], _p64(rp), _p32(ci)))



def _u8p(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8))


def kcore_members(rowptr, colidx, k: int):
    """uint8 mask of the k-core, by repeated deletion of degree < k."""
    rp, ci, n = _csr(rowptr, colidx)
    mask = np.empty(max(n, 1), dtype=np.uint8)
    if _load().oracle_kcore_members(n, _p64(rp), _p32(ci), int(k), _u8p(mask)) != 0:
        raise RuntimeError("oracle_kcore_members failed")
    return mask[:n]


def induced_csr(rowptr, colidx, keep):
    """(rowptr, colidx, vmap) of G[{v: keep[v]}], renumbered by increasing id."""
    rp, ci, n = _csr(rowptr, colidx)
    kp = np.ascontiguousarray(np.asarray(keep), dtype=np.uint8)
    nk, mk = ctypes.c_int64(0), ctypes.c_int64(0)
    lib = _load()
    lib.oracle_induced_csr(n, _p64(rp), _p32(ci), _u8p(kp), ctypes.byref(nk), ctypes.byref(mk), None, None, None)
    orp = np.zeros(nk.value + 1, dtype=np.int64)
    oci = np.empty(max(mk.value, 1), dtype=np.int32)
    vm = np.empty(max(nk.value, 1), dtype=np.int32)
    lib.oracle_induced_csr(n, _p64(rp), _p32(ci), _u8p(kp), ctypes.byref(nk), ctypes.byref(mk), _p64(orp),
                           _p32(oci), _p32(vm))
    return orp, oci[:mk.value], vm[:nk.value]


def mpm(rowptr, colidx, max_iters: int = -1):
    """Synchronous MPM: (a, iterations).  a = core at convergence."""
    rp, ci, n = _csr(rowptr, colidx)
    a = np.empty(max(n, 1), dtype=np.int32)
    it = ctypes.c_int64(0)
    if _load().oracle_mpm(n, _p64(rp), _p32(ci), int(max_iters), _p32(a), ctypes.byref(it)) != 0:
        raise RuntimeError("oracle_mpm failed")
    return a[:n], int(it.value)
