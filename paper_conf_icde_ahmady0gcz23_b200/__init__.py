"""B200-native k-core decomposition (Ahmad et al., ICDE 2023 -- PAPER.md).

Thin Python binding over the C ABI in ``include/kcore.h`` (library
``lib/libkcore.so``, built in-tree by ``make``).  Argument marshalling only:
every step of the decomposition runs in the library's sm_100a kernels.  PyTorch
supplies device memory, streams and process groups.  There is no CPU fallback:
if the library is missing or the device is not a B200 every call raises.

Entry points mirror the C names:

* :func:`kcore_decompose`       -- core numbers of a CSR graph on one GPU.
* :func:`kcore_decompose_host`  -- same from/to host buffers (end-to-end path).
* :func:`kcore_decompose_mg`    -- multi-GPU, 1-D vertex-range ownership (NCCL).
* :func:`kcore_decompose_mg_virtual` -- the multi-GPU protocol with virtual
  ranks on one GPU (testing).
* :func:`kcore_kshell`, :func:`kcore_kcore_mask`, :func:`kcore_kcore_subgraph` -- k-shell /
  k-core outputs of a decomposition.
* :func:`kcore_mpm`             -- the MPM h-index iteration (the paper's second family).
* :func:`kcore_validate_csr`, :func:`kcore_workspace_size`, :func:`kcore_strerror`.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("KCORE_LIB") or os.path.join(_HERE, "lib", "libkcore.so")  # override: tuning sweeps

KCORE_OK = 0
KCORE_EINVAL = -1
KCORE_ENOMEM = -2
KCORE_ECUDA = -3
KCORE_ENCCL = -4
KCORE_EGRAPH = -5
KCORE_EUNSUPPORTED = -6

ALGO_PERSISTENT = 0
ALGO_HOSTLOOP = 1
FLAG_NO_BLOOM = 1
FLAG_NO_L2_PERSIST = 2
FLAG_NO_RED = 4
FLAG_NO_NEAR = 8

# every symbol include/kcore.h declares (checked by tests/test_abi.py)
EXPORTS = (
    "kcore_decompose", "kcore_decompose_ex", "kcore_decompose_host", "kcore_workspace_size",
    "kcore_validate_csr", "kcore_strerror", "kcore_version", "kcore_decompose_mg",
    "kcore_decompose_mg_virtual", "kcore_nccl_unique_id", "kcore_nccl_comm_init",
    "kcore_nccl_comm_destroy", "kcore_kshell", "kcore_kcore_mask", "kcore_kcore_subgraph", "kcore_mpm",
    "kcore_decompose_mg_ex", "kcore_decompose_mg_virtual_ex",
)


class KcoreError(RuntimeError):
    def __init__(self, status: int, what: str):
        self.status = status
        super().__init__(f"{what}: {strerror(status)} ({status})")


class _Options(ctypes.Structure):
    _fields_ = [
        ("algo", ctypes.c_int32), ("blocks_per_sm", ctypes.c_int32),
        ("solo_arcs", ctypes.c_int32), ("solo_scan", ctypes.c_int32),
        ("order_out", ctypes.c_void_p), ("workspace", ctypes.c_void_p),
        ("workspace_bytes", ctypes.c_size_t), ("trace_out", ctypes.c_void_p),
        ("trace_cap", ctypes.c_int64), ("flags", ctypes.c_int32), ("reserved1", ctypes.c_int32),
        ("trace_cta_out", ctypes.c_void_p), ("near_min_alive", ctypes.c_int32), ("near_window", ctypes.c_int32),
    ]


class _Stats(ctypes.Structure):
    _fields_ = [
        ("levels", ctypes.c_int64), ("phases", ctypes.c_int64),
        ("solo_phases", ctypes.c_int64), ("barriers", ctypes.c_int64),
        ("scanned", ctypes.c_int64), ("arcs_walked", ctypes.c_int64),
        ("compactions", ctypes.c_int64), ("hub_arcs", ctypes.c_int64), ("kmax", ctypes.c_int32),
        ("grid_blocks", ctypes.c_int32), ("block_threads", ctypes.c_int32),
        ("trace_len", ctypes.c_int32), ("kernel_ms", ctypes.c_double),
        ("launches", ctypes.c_int64), ("near_scans", ctypes.c_int64), ("reserved", ctypes.c_int64 * 1),
    ]


@dataclass
class Stats:
    levels: int
    phases: int
    solo_phases: int
    barriers: int
    scanned: int
    arcs_walked: int
    compactions: int
    hub_arcs: int
    kmax: int
    grid_blocks: int
    block_threads: int
    kernel_ms: float
    trace_len: int = 0
    launches: int = 0
    near_scans: int = 0

    @classmethod
    def _from(cls, s: _Stats) -> "Stats":
        return cls(s.levels, s.phases, s.solo_phases, s.barriers, s.scanned, s.arcs_walked,
                   s.compactions, s.hub_arcs, s.kmax, s.grid_blocks, s.block_threads, s.kernel_ms,
                   s.trace_len, s.launches, s.near_scans)


_lib = None


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: build it with `make` (__graft_entry__.build()); "
                               "there is no CPU fallback")
        import torch  # noqa: F401  (loads torch's libnccl.so.2 first so both share one copy)
        lib = ctypes.CDLL(LIB_PATH)
        vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
        lib.kcore_decompose.argtypes = [vp, vp, i64, i64, vp, vp]
        lib.kcore_decompose_ex.argtypes = [vp, vp, i64, i64, vp, vp, ctypes.POINTER(_Options),
                                           ctypes.POINTER(_Stats)]
        lib.kcore_decompose_host.argtypes = [vp, vp, i64, i64, vp, vp, ctypes.POINTER(_Options),
                                             ctypes.POINTER(_Stats)]
        lib.kcore_workspace_size.argtypes = [i64, i64]
        lib.kcore_workspace_size.restype = ctypes.c_size_t
        lib.kcore_validate_csr.argtypes = [vp, vp, i64, i64, vp]
        lib.kcore_strerror.argtypes = [ctypes.c_int]
        lib.kcore_strerror.restype = ctypes.c_char_p
        lib.kcore_version.restype = ctypes.c_char_p
        lib.kcore_decompose_mg.argtypes = [vp, vp, i64, i64, i64, i64, vp, vp, vp, ctypes.POINTER(_Stats)]
        lib.kcore_decompose_mg_virtual.argtypes = [vp, vp, i64, i64, i32, vp, vp, ctypes.POINTER(_Stats)]
        lib.kcore_decompose_mg_ex.argtypes = [vp, vp, i64, i64, i64, i64, vp, vp, vp, i32, ctypes.POINTER(_Stats)]
        lib.kcore_decompose_mg_virtual_ex.argtypes = [vp, vp, i64, i64, i32, vp, vp, i32, ctypes.POINTER(_Stats)]
        lib.kcore_nccl_unique_id.argtypes = [vp]
        lib.kcore_nccl_comm_init.argtypes = [ctypes.POINTER(vp), i32, vp, i32]
        lib.kcore_nccl_comm_destroy.argtypes = [vp]
        i64p = ctypes.POINTER(ctypes.c_int64)
        lib.kcore_kshell.argtypes = [vp, i64, i32, vp, i64p, vp]
        lib.kcore_kcore_mask.argtypes = [vp, i64, i32, vp, i64p, vp]
        lib.kcore_kcore_subgraph.argtypes = [vp, vp, vp, i64, i64, i32, i64p, i64p, vp, vp, vp, vp]
        lib.kcore_mpm.argtypes = [vp, vp, i64, i64, vp, i64, i64p, vp, ctypes.POINTER(_Stats)]
        _lib = lib
    return _lib


def library():
    """The loaded ctypes handle (raises if the library is missing)."""
    return _load()


def strerror(status: int) -> str:
    try:
        return _load().kcore_strerror(status).decode()
    except RuntimeError:
        return f"status {status}"


def version() -> str:
    return _load().kcore_version().decode()


def kcore_workspace_size(n: int, m: int = 0) -> int:
    return int(_load().kcore_workspace_size(n, m))


def _stream_ptr(device):
    import torch
    return torch.cuda.current_stream(device).cuda_stream


def _check_csr_tensors(rowptr, colidx):
    import torch
    if not (rowptr.is_cuda and colidx.is_cuda):
        raise ValueError("rowptr/colidx must be CUDA tensors (use kcore_decompose_host for host buffers)")
    if rowptr.dtype != torch.int64 or colidx.dtype != torch.int32:
        raise TypeError("rowptr must be int64 and colidx int32")
    if not (rowptr.is_contiguous() and colidx.is_contiguous()):
        raise ValueError("rowptr/colidx must be contiguous")
    if rowptr.device != colidx.device:
        raise ValueError("rowptr/colidx on different devices")


def kcore_decompose(rowptr, colidx, *, core_out=None, order_out=None, workspace=None,
                    algo: int = ALGO_PERSISTENT, blocks_per_sm: int = 0, solo_arcs: int = 0,
                    solo_scan: int = 0, bloom: bool = True, trace=None,
                    trace_cta=None, stats: bool = False, l2_persist: bool = True, red: bool = True,
                    near: bool = True, near_min_alive: int = 0, near_window: int = 0):
    """Core numbers of the graph (rowptr int64[n+1], colidx int32[m] CUDA tensors).

    Runs on the current stream of the tensors' device.  Returns an int32 tensor
    ``core`` (and a :class:`Stats` if ``stats=True``, which synchronises)."""
    import torch
    _check_csr_tensors(rowptr, colidx)
    dev = rowptr.device
    n = rowptr.numel() - 1
    m = colidx.numel()
    if core_out is None:
        core_out = torch.empty(max(n, 0), dtype=torch.int32, device=dev)
    opt = _Options(algo, blocks_per_sm, solo_arcs, solo_scan,
                   order_out.data_ptr() if order_out is not None else None,
                   workspace.data_ptr() if workspace is not None else None,
                   workspace.numel() * workspace.element_size() if workspace is not None else 0,
                   trace.data_ptr() if trace is not None else None,
                   trace.shape[0] if trace is not None else 0,
                   (0 if bloom else FLAG_NO_BLOOM) | (0 if l2_persist else FLAG_NO_L2_PERSIST) |
                   (0 if red else FLAG_NO_RED) | (0 if near else FLAG_NO_NEAR), 0,
                   trace_cta.data_ptr() if trace_cta is not None else None, near_min_alive, near_window)
    st = _Stats()
    with torch.cuda.device(dev):
        rc = _load().kcore_decompose_ex(rowptr.data_ptr(), colidx.data_ptr() if m else None, n, m,
                                        core_out.data_ptr() if n else None, _stream_ptr(dev),
                                        ctypes.byref(opt), ctypes.byref(st) if stats else None)
    if rc != KCORE_OK:
        raise KcoreError(rc, "kcore_decompose")
    return (core_out, Stats._from(st)) if stats else core_out


def kcore_decompose_host(rowptr, colidx, *, core_out=None, stats: bool = False, device=None,
                         algo: int = ALGO_PERSISTENT):
    """End-to-end: host (ideally pinned) int64/int32 tensors in, host int32 core out."""
    import torch
    if rowptr.is_cuda or colidx.is_cuda:
        raise ValueError("kcore_decompose_host takes host tensors")
    if rowptr.dtype != torch.int64 or colidx.dtype != torch.int32:
        raise TypeError("rowptr must be int64 and colidx int32")
    dev = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
    n = rowptr.numel() - 1
    m = colidx.numel()
    if core_out is None:
        core_out = torch.empty(max(n, 0), dtype=torch.int32, pin_memory=rowptr.is_pinned())
    opt = _Options(algo, 0, 0, 0, None, None, 0, None, 0)
    st = _Stats()
    with torch.cuda.device(dev):
        rc = _load().kcore_decompose_host(rowptr.data_ptr(), colidx.data_ptr() if m else None, n, m,
                                          core_out.data_ptr() if n else None, _stream_ptr(dev),
                                          ctypes.byref(opt), ctypes.byref(st) if stats else None)
    if rc != KCORE_OK:
        raise KcoreError(rc, "kcore_decompose_host")
    return (core_out, Stats._from(st)) if stats else core_out


def kcore_validate_csr(rowptr, colidx) -> int:
    """KCORE_OK if the CUDA CSR satisfies the preconditions, else KCORE_EGRAPH."""
    import torch
    _check_csr_tensors(rowptr, colidx)
    n = rowptr.numel() - 1
    m = colidx.numel()
    with torch.cuda.device(rowptr.device):
        rc = _load().kcore_validate_csr(rowptr.data_ptr(), colidx.data_ptr() if m else None, n, m,
                                        _stream_ptr(rowptr.device))
    if rc not in (KCORE_OK, KCORE_EGRAPH):
        raise KcoreError(rc, "kcore_validate_csr")
    return rc


def kcore_decompose_mg_virtual(rowptr, colidx, nranks: int, *, stats: bool = False, algo: int = 0):
    """Multi-GPU protocol with `nranks` virtual ranks on this GPU (global CSR in, global core out).
    algo 0 (KCORE_MG_DEVICE): the device-initiated kernel; 1 (KCORE_MG_HOSTLOOP): host-driven."""
    import torch
    _check_csr_tensors(rowptr, colidx)
    dev = rowptr.device
    n = rowptr.numel() - 1
    m = colidx.numel()
    core = torch.empty(max(n, 0), dtype=torch.int32, device=dev)
    st = _Stats()
    with torch.cuda.device(dev):
        rc = _load().kcore_decompose_mg_virtual_ex(rowptr.data_ptr(), colidx.data_ptr() if m else None, n, m,
                                                   nranks, core.data_ptr() if n else None, _stream_ptr(dev),
                                                   int(algo), ctypes.byref(st) if stats else None)
    if rc != KCORE_OK:
        raise KcoreError(rc, "kcore_decompose_mg_virtual")
    return (core, Stats._from(st)) if stats else core


def _check_core(core):
    import torch
    if not core.is_cuda or core.dtype != torch.int32 or not core.is_contiguous():
        raise TypeError("core must be a contiguous int32 CUDA tensor")


def kcore_kshell(core, k: int):
    """The k-shell {v : core[v] == k} as an int32 CUDA tensor of vertex ids (increasing)."""
    import torch
    _check_core(core)
    n = core.numel()
    cnt = ctypes.c_int64(0)
    lib = _load()
    with torch.cuda.device(core.device):
        rc = lib.kcore_kshell(core.data_ptr() if n else None, n, int(k), None, ctypes.byref(cnt),
                              _stream_ptr(core.device))
        if rc != KCORE_OK:
            raise KcoreError(rc, "kcore_kshell")
        out = torch.empty(cnt.value, dtype=torch.int32, device=core.device)
        if cnt.value:
            rc = lib.kcore_kshell(core.data_ptr(), n, int(k), out.data_ptr(), ctypes.byref(cnt),
                                  _stream_ptr(core.device))
            if rc != KCORE_OK:
                raise KcoreError(rc, "kcore_kshell")
    return out


def kcore_kcore_mask(core, k: int):
    """(uint8 CUDA mask of the k-core {v : core[v] >= k}, its size)."""
    import torch
    _check_core(core)
    n = core.numel()
    mask = torch.empty(n, dtype=torch.uint8, device=core.device)
    cnt = ctypes.c_int64(0)
    with torch.cuda.device(core.device):
        rc = _load().kcore_kcore_mask(core.data_ptr() if n else None, n, int(k), mask.data_ptr() if n else None,
                                      ctypes.byref(cnt), _stream_ptr(core.device))
    if rc != KCORE_OK:
        raise KcoreError(rc, "kcore_kcore_mask")
    return mask, int(cnt.value)


def kcore_kcore_subgraph(rowptr, colidx, core, k: int):
    """The induced k-core subgraph: (sub_rowptr int64, sub_colidx int32, vmap int32) CUDA
    tensors, vertices renumbered in increasing original id (vmap[new] = old)."""
    import torch
    _check_csr_tensors(rowptr, colidx)
    _check_core(core)
    n = rowptr.numel() - 1
    m = colidx.numel()
    nk, mk = ctypes.c_int64(0), ctypes.c_int64(0)
    lib = _load()
    dev = rowptr.device
    cp = colidx.data_ptr() if m else None
    with torch.cuda.device(dev):
        rc = lib.kcore_kcore_subgraph(rowptr.data_ptr(), cp, core.data_ptr() if n else None, n, m, int(k),
                                      ctypes.byref(nk), ctypes.byref(mk), None, None, None, _stream_ptr(dev))
        if rc != KCORE_OK:
            raise KcoreError(rc, "kcore_kcore_subgraph")
        srp = torch.empty(nk.value + 1, dtype=torch.int64, device=dev)
        sci = torch.empty(max(mk.value, 1), dtype=torch.int32, device=dev)
        vm = torch.empty(max(nk.value, 1), dtype=torch.int32, device=dev)
        rc = lib.kcore_kcore_subgraph(rowptr.data_ptr(), cp, core.data_ptr() if n else None, n, m, int(k),
                                      ctypes.byref(nk), ctypes.byref(mk), srp.data_ptr(), sci.data_ptr(),
                                      vm.data_ptr(), _stream_ptr(dev))
    if rc != KCORE_OK:
        raise KcoreError(rc, "kcore_kcore_subgraph")
    return srp, sci[:mk.value], vm[:nk.value]


def kcore_mpm(rowptr, colidx, *, max_iters: int = -1, a_out=None, stats: bool = False):
    """MPM h-index iteration (bulk-synchronous as P:L388): (a, iterations[, Stats]).
    a = core at convergence; with max_iters >= 0, the iterate after that many iterations."""
    import torch
    _check_csr_tensors(rowptr, colidx)
    dev = rowptr.device
    n = rowptr.numel() - 1
    m = colidx.numel()
    if a_out is None:
        a_out = torch.empty(max(n, 0), dtype=torch.int32, device=dev)
    it = ctypes.c_int64(0)
    st = _Stats()
    with torch.cuda.device(dev):
        rc = _load().kcore_mpm(rowptr.data_ptr(), colidx.data_ptr() if m else None, n, m,
                               a_out.data_ptr() if n else None, int(max_iters), ctypes.byref(it),
                               _stream_ptr(dev), ctypes.byref(st) if stats else None)
    if rc != KCORE_OK:
        raise KcoreError(rc, "kcore_mpm")
    return (a_out, int(it.value), Stats._from(st)) if stats else (a_out, int(it.value))


from .parallel import (  # noqa: E402
    NcclComm, kcore_decompose_mg, owner_ranges, local_csr, gather_cores,
)

__all__ = [
    "kcore_decompose", "kcore_decompose_host", "kcore_decompose_mg", "kcore_decompose_mg_virtual",
    "kcore_validate_csr", "kcore_workspace_size", "strerror", "version", "Stats", "KcoreError",
    "NcclComm", "owner_ranges", "local_csr", "gather_cores", "EXPORTS", "LIB_PATH",
    "kcore_kshell", "kcore_kcore_mask", "kcore_kcore_subgraph", "kcore_mpm",
]
