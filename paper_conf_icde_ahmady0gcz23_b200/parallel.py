"""Multi-GPU plumbing around ``kcore_decompose_mg`` (include/kcore.h).

1-D vertex-range ownership (north star; the paper's multi-GPU future work,
P:L587, routed to owners instead of a master GPU): rank r of P owns vertices
``[r*n//P, (r+1)*n//P)`` and stores their CSR rows with global neighbour ids.
This module holds the host-side logic only -- range computation, slicing a
global CSR into a rank's rows, NCCL communicator setup over a
``torch.distributed`` group, and gathering per-rank results -- all of which is
exercised by world_size-2 gloo tests on CPU.  The decomposition itself runs in
the library's kernels with NCCL between GPUs.
"""
from __future__ import annotations

import ctypes

KCORE_OK = 0


def owner_ranges(n: int, nranks: int):
    """[(v_begin, v_end)] for every rank: equal contiguous ranges tiling [0, n)."""
    if nranks < 1:
        raise ValueError("nranks >= 1")
    b = [(r * n) // nranks for r in range(nranks + 1)]
    return [(b[r], b[r + 1]) for r in range(nranks)]


def owner_of(v: int, n: int, nranks: int) -> int:
    """Rank owning global vertex v under owner_ranges (the routing rule of the
    decrement exchange; mirrored by the device code's owner lookup)."""
    r = (v * nranks) // n if n else 0
    # floor-division ranges can put v one rank off the estimate
    while r > 0 and v < (r * n) // nranks:
        r -= 1
    while r + 1 < nranks and v >= ((r + 1) * n) // nranks:
        r += 1
    return r


def local_csr(rowptr, colidx, v_begin: int, v_end: int):
    """A rank's rows of a global CSR: (local rowptr with offsets from 0, colidx
    with global ids).  Works on numpy arrays and torch tensors alike."""
    a0 = int(rowptr[v_begin])
    a1 = int(rowptr[v_end])
    return rowptr[v_begin:v_end + 1] - a0, colidx[a0:a1]


def gather_cores(core_local, group=None):
    """Concatenate every rank's core_out_local (in rank order) on all ranks."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    sizes = [None] * world
    dist.all_gather_object(sizes, int(core_local.numel()), group=group)
    mx = max(sizes)
    buf = torch.zeros(mx, dtype=core_local.dtype, device=core_local.device)
    buf[: core_local.numel()] = core_local
    outs = [torch.empty_like(buf) for _ in range(world)]
    dist.all_gather(outs, buf, group=group)
    return torch.cat([o[:s] for o, s in zip(outs, sizes)])


class NcclComm:
    """An NCCL communicator owned by libkcore, set up over a torch.distributed
    group: rank 0 draws the unique id, the group broadcasts it (gloo or NCCL)."""

    def __init__(self, group=None, device=None):
        import torch
        import torch.distributed as dist
        from . import _load
        self._lib = _load()
        self.rank = dist.get_rank(group)
        self.size = dist.get_world_size(group)
        raw = ctypes.create_string_buffer(128)
        if self.rank == 0:
            rc = self._lib.kcore_nccl_unique_id(raw)
            if rc != KCORE_OK:
                raise RuntimeError(f"kcore_nccl_unique_id: {rc}")
        obj = [bytes(raw.raw) if self.rank == 0 else None]
        dist.broadcast_object_list(obj, src=dist.get_global_rank(group, 0) if group is not None else 0,
                                   group=group)
        idbuf = ctypes.create_string_buffer(obj[0], 128)
        dev = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
        self.handle = ctypes.c_void_p()
        with torch.cuda.device(dev):
            rc = self._lib.kcore_nccl_comm_init(ctypes.byref(self.handle), self.size, idbuf, self.rank)
        if rc != KCORE_OK:
            raise RuntimeError(f"kcore_nccl_comm_init: {rc}")

    def close(self):
        if self.handle:
            self._lib.kcore_nccl_comm_destroy(self.handle)
            self.handle = ctypes.c_void_p()

    def __del__(self):  # pragma: no cover
        try:
            self.close()
        except Exception:
            pass


MG_DEVICE = 0    # device-initiated persistent kernel over NCCL symmetric windows
MG_HOSTLOOP = 1  # host-driven NCCL exchange per sub-round (default of kcore_decompose_mg)


def kcore_decompose_mg(rowptr_local, colidx_local, n_global: int, v_begin: int, v_end: int,
                       comm: NcclComm, *, stats: bool = False, algo: int = MG_HOSTLOOP):
    """This rank's core numbers (int32 CUDA tensor of v_end-v_begin entries).
    Collective over `comm`.  algo=MG_HOSTLOOP synchronises the stream per
    sub-round; algo=MG_DEVICE runs one persistent kernel per rank."""
    import torch
    from . import KcoreError, Stats, _Stats, _check_csr_tensors, _load, _stream_ptr
    _check_csr_tensors(rowptr_local, colidx_local)
    dev = rowptr_local.device
    nl = v_end - v_begin
    if rowptr_local.numel() != nl + 1:
        raise ValueError("rowptr_local must have v_end - v_begin + 1 entries")
    core = torch.empty(max(nl, 0), dtype=torch.int32, device=dev)
    st = _Stats()
    m_local = colidx_local.numel()
    with torch.cuda.device(dev):
        rc = _load().kcore_decompose_mg_ex(rowptr_local.data_ptr(), colidx_local.data_ptr() if m_local else None,
                                           n_global, v_begin, v_end, m_local,
                                           core.data_ptr() if nl else None, _stream_ptr(dev), comm.handle,
                                           int(algo), ctypes.byref(st) if stats else None)
    if rc != KCORE_OK:
        raise KcoreError(rc, "kcore_decompose_mg")
    return (core, Stats._from(st)) if stats else core
