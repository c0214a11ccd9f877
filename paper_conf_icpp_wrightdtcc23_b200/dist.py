"""a12: row-partitioned multi-GPU SpMV, one process per GPU (north_star; the
paper itself is single-GPU).

torch.distributed is the plumbing: it broadcasts the 128-byte NCCL unique id
that libnest.so's communicator is built from.  The all-gather of x and the
local SpMV run inside libnest.so (``nest_spmv_csr_f64_dist``), on the caller's
stream.
"""
from __future__ import annotations

import ctypes

from . import _nest as N
from .api import _dev, _stream, _torch, check, make_desc


def shard_rows(n: int, nranks: int, rank: int):
    """Equal-row partition: chunk = ceil(n/P); rank r owns
    [r*chunk, min((r+1)*chunk, n)).  Returns (chunk, row_begin, nrows_local)."""
    if nranks <= 0 or not 0 <= rank < nranks or n < 0:
        raise ValueError("bad partition arguments")
    chunk = -(-n // nranks)
    b = min(rank * chunk, n)
    return chunk, b, min(b + chunk, n) - b


def x_chunk(ncols: int, nranks: int) -> int:
    """x is all-gathered in equal chunks of ceil(ncols/P) doubles, so global
    column j lands at x_full[j] (x_full holds P*xchunk doubles)."""
    return -(-ncols // nranks)


def local_x_range(ncols: int, nranks: int, rank: int):
    """(begin, count) of the slice of x that rank owns; the tail rank pads."""
    xc = x_chunk(ncols, nranks)
    b = min(rank * xc, ncols)
    return b, min(xc, ncols - b)


def broadcast_unique_id(group=None) -> bytes:
    """Rank 0 creates the 128-byte NCCL unique id inside libnest.so; the torch
    process group (any backend) broadcasts it to every rank."""
    import torch.distributed as dist
    uid = (ctypes.c_uint8 * 128)()
    if dist.get_rank(group) == 0:
        check(N.nest_comm_unique_id(uid), "nest_comm_unique_id")
    obj = [bytes(uid)]
    src = 0 if group is None else dist.get_global_rank(group, 0)
    dist.broadcast_object_list(obj, src=src, group=group)
    return obj[0]


class Comm:
    """A libnest-owned NCCL communicator over the ranks of a torch process group."""

    def __init__(self, group=None):
        torch = _torch()
        import torch.distributed as dist
        self.rank = dist.get_rank(group)
        self.nranks = dist.get_world_size(group)
        uid = (ctypes.c_uint8 * 128).from_buffer_copy(broadcast_unique_id(group))
        self._h = ctypes.c_void_p()
        check(N.nest_comm_init(uid, self.nranks, self.rank, ctypes.byref(self._h)), "nest_comm_init")
        self._torch = torch

    def close(self):
        if self._h:
            check(N.nest_comm_destroy(self._h), "nest_comm_destroy")
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def spmv_csr_f64(self, nrows_global, ncols_global, rowptr, colind, val, x_local, x_full,
                     y_local=None, *, stream=None, **cfg):
        """y_local = A[local rows] @ x after all-gathering x (x_full is scratch/output)."""
        torch = self._torch
        nrows_local = rowptr.numel() - 1
        nnz = val.numel()
        xchunk = x_chunk(ncols_global, self.nranks)
        if y_local is None:
            y_local = torch.empty(nrows_local, dtype=torch.float64, device=val.device)
        d = make_desc(**cfg)
        check(N.nest_spmv_csr_f64_dist(ctypes.byref(d), self._h, nrows_global, ncols_global,
                                       nrows_local, nnz,
                                       _dev(rowptr, torch.int64, nrows_local + 1, "rowptr"),
                                       _dev(colind, torch.int32, nnz, "colind"),
                                       _dev(val, torch.float64, nnz, "val"),
                                       _dev(x_local, torch.float64, xchunk, "x_local"),
                                       _dev(x_full, torch.float64, xchunk * self.nranks, "x_full"),
                                       _dev(y_local, torch.float64, nrows_local, "y_local"),
                                       _stream(stream)),
              "nest_spmv_csr_f64_dist")
        return y_local


    def allgather_x(self, x_local, x_full, ncols_global, *, stream=None):
        """a12's exchange step alone: x_full = all ranks' x_local slices."""
        torch = self._torch
        xc = x_chunk(ncols_global, self.nranks)
        check(N.nest_comm_allgather_x(self._h, _dev(x_local, torch.float64, xc, "x_local"),
                                      _dev(x_full, torch.float64, xc * self.nranks, "x_full"), xc,
                                      _stream(stream)), "nest_comm_allgather_x")
        return x_full

    def hostio_workspace_bytes(self, nrows_local, nnz_local, ncols_global) -> int:
        return int(N.nest_spmv_dist_hostio_workspace_bytes(nrows_local, nnz_local,
                                                           x_chunk(ncols_global, self.nranks), self.nranks))

    def spmv_csr_f64_hostio(self, nrows_global, ncols_global, h_rowptr, h_colind, h_val, h_x_local, h_y,
                            workspace, *, stream=None, **cfg):
        """a12 end to end: HOST (pinned) shard and x slice in, y_local out."""
        torch = self._torch
        nrows_local = h_rowptr.numel() - 1
        nnz = h_val.numel()
        xc = x_chunk(ncols_global, self.nranks)
        for t, dt, name, n in ((h_rowptr, torch.int64, "h_rowptr", nrows_local + 1),
                               (h_colind, torch.int32, "h_colind", nnz), (h_val, torch.float64, "h_val", nnz),
                               (h_x_local, torch.float64, "h_x_local", xc), (h_y, torch.float64, "h_y", nrows_local)):
            if t.is_cuda or t.dtype != dt or not t.is_contiguous():
                raise TypeError(f"{name} must be a contiguous host {dt} tensor")
            if t.numel() < n:
                raise ValueError(f"{name} has {t.numel()} elements, needs {n}")
        d = make_desc(**cfg)
        check(N.nest_spmv_csr_f64_dist_hostio(ctypes.byref(d), self._h, nrows_global, ncols_global, nrows_local, nnz,
                                              ctypes.c_void_p(h_rowptr.data_ptr()),
                                              ctypes.c_void_p(h_colind.data_ptr()),
                                              ctypes.c_void_p(h_val.data_ptr()),
                                              ctypes.c_void_p(h_x_local.data_ptr()),
                                              ctypes.c_void_p(h_y.data_ptr()),
                                              _dev(workspace, torch.uint8, None, "workspace"), workspace.numel(),
                                              _stream(stream)), "nest_spmv_csr_f64_dist_hostio")
        return h_y


class XPeer:
    """NEXT-4: comm-free row-partitioned SpMV.  x stays distributed: this rank's
    slice lives in a libnest-owned buffer every peer maps (CUDA IPC), and the
    SpMV's simd lanes gather x[c] from the owner's slice over NVLink -- no
    all-gather.  torch.distributed only exchanges the IPC handle blobs.

    ``local_slices``: single-process form (tests): a list of nranks CUDA tensors
    (xchunk doubles each) standing for the ranks' slices; no IPC, no barrier."""

    def __init__(self, ncols_global: int, group=None, *, nranks=None, rank=None, local_slices=None):
        torch = _torch()
        self._torch = torch
        self._h = ctypes.c_void_p()
        if local_slices is not None:
            self.nranks, self.rank = int(nranks), int(rank)
            xc = x_chunk(ncols_global, self.nranks)
            if len(local_slices) != self.nranks:
                raise ValueError("need one slice per rank")
            arr = (ctypes.c_void_p * self.nranks)(*[_dev(t, torch.float64, xc, f"slice {r}").value if xc else None
                                                    for r, t in enumerate(local_slices)])
            self._keep = list(local_slices)
            check(N.nest_xpeer_create_local(self.nranks, self.rank, ncols_global, arr, ctypes.byref(self._h)),
                  "nest_xpeer_create_local")
            return
        import torch.distributed as dist
        self.rank = dist.get_rank(group)
        self.nranks = dist.get_world_size(group)
        nb = int(N.nest_xpeer_handle_bytes())
        blob = (ctypes.c_uint8 * nb)()
        check(N.nest_xpeer_create(self.nranks, self.rank, ncols_global, ctypes.byref(self._h), blob),
              "nest_xpeer_create")
        blobs = [None] * self.nranks
        dist.all_gather_object(blobs, bytes(blob), group=group)
        allb = (ctypes.c_uint8 * (nb * self.nranks)).from_buffer_copy(b"".join(blobs))
        check(N.nest_xpeer_open(self._h, allb), "nest_xpeer_open")

    @property
    def xchunk(self) -> int:
        return int(N.nest_xpeer_xchunk(self._h))

    def local_x(self):
        """This rank's x slice (library-owned device memory) as a borrowed pointer."""
        return N.nest_xpeer_local_x(self._h)

    def set_local_x(self, x_local, stream=None):
        """Copy this rank's part of x (a CUDA tensor, >= its slice length) into
        its library-owned slice, stream-ordered (device to device)."""
        torch = self._torch
        check(N.nest_xpeer_set_x(self._h, _dev(x_local, torch.float64, None, "x_local"), x_local.numel(),
                                 _stream(stream)), "nest_xpeer_set_x")

    def barrier(self, stream=None):
        check(N.nest_xpeer_barrier(self._h, _stream(stream)), "nest_xpeer_barrier")

    def spmv_csr_f64(self, nrows_global, rowptr, colind, val, y_local=None, *, stream=None, **cfg):
        """barrier; y_local = A[local rows] @ x gathering x from the owners' slices; barrier."""
        torch = self._torch
        nrows_local = rowptr.numel() - 1
        nnz = val.numel()
        if y_local is None:
            y_local = torch.empty(nrows_local, dtype=torch.float64, device=val.device)
        d = make_desc(**cfg)
        check(N.nest_spmv_csr_f64_xpeer(ctypes.byref(d), self._h, nrows_global, nrows_local, nnz,
                                        _dev(rowptr, torch.int64, nrows_local + 1, "rowptr"),
                                        _dev(colind, torch.int32, nnz, "colind"),
                                        _dev(val, torch.float64, nnz, "val"),
                                        _dev(y_local, torch.float64, nrows_local, "y_local"),
                                        _stream(stream)),
              "nest_spmv_csr_f64_xpeer")
        return y_local

    def close(self):
        if self._h:
            check(N.nest_xpeer_destroy(self._h), "nest_xpeer_destroy")
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _exchange_fds(fd: int, rank: int, nranks: int, tag: str, group=None) -> list:
    """Every rank's file descriptor to every rank (SCM_RIGHTS over unix sockets on this
    node; torch.distributed only orders the steps).  Returns a list of nranks fds
    (the entry at `rank` is `fd` itself)."""
    import os
    import socket
    import threading

    import torch.distributed as dist
    path = lambda r: f"/tmp/nest_xsym_{tag}_{r}.sock"   # noqa: E731
    me = path(rank)
    if os.path.exists(me):
        os.unlink(me)
    srv = socket.socket(socket.AF_UNIX, socket.SOCK_STREAM)
    srv.bind(me)
    srv.listen(nranks)
    got = {rank: fd}

    def serve():
        for _ in range(nranks - 1):
            conn, _ = srv.accept()
            with conn:
                msg, fds, _, _ = socket.recv_fds(conn, 16, 1)
                got[int(msg.decode())] = fds[0]
    t = threading.Thread(target=serve, daemon=True)
    t.start()
    dist.barrier(group=group)                 # every rank listens
    for r in range(nranks):
        if r != rank:
            with socket.socket(socket.AF_UNIX, socket.SOCK_STREAM) as c:
                c.connect(path(r))
                socket.send_fds(c, [str(rank).encode()], [fd])
    t.join()
    srv.close()
    dist.barrier(group=group)                 # every rank has every descriptor
    os.unlink(me)
    return [got[r] for r in range(nranks)]


class XSym:
    """NEXT-4b: x as ONE virtual range over every rank's slice (CUDA virtual memory,
    POSIX file descriptors exchanged on this node).  ``x`` is the contiguous global x
    (column j at x[j] on every rank), so the row-partitioned SpMV is the ordinary
    ``spmv_csr_f64(rowptr_local, colind_global, val, xs.x(), ...)`` -- any variant.
    ``nranks`` without a process group: single-process form, every slice local."""

    def __init__(self, ncols_global: int, group=None, *, nranks=None, tag="x"):
        import os
        torch = _torch()
        self._torch = torch
        self._h = ctypes.c_void_p()
        self.ncols = int(ncols_global)
        if nranks is not None:
            self.nranks, self.rank = int(nranks), 0
            check(N.nest_xsym_create_local(self.nranks, self.ncols, ctypes.byref(self._h)),
                  "nest_xsym_create_local")
            return
        import torch.distributed as dist
        self.rank, self.nranks = dist.get_rank(group), dist.get_world_size(group)

        def all_ok(status):   # every rank agrees before the next collective step
            dev = "cuda" if dist.get_backend(group) == "nccl" else "cpu"
            t = torch.tensor([1 if status == N.NEST_OK else 0], dtype=torch.int32, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
            return int(t.item()) == 1

        fd = ctypes.c_int32(-1)
        st = N.nest_xsym_create(self.nranks, self.rank, self.ncols, ctypes.byref(self._h), ctypes.byref(fd))
        if not all_ok(st):
            if fd.value >= 0:
                os.close(fd.value)
            self.close()
            check(st if st != N.NEST_OK else N.NEST_ERR_CUDA, "nest_xsym_create (on some rank)")
        fds = _exchange_fds(fd.value, self.rank, self.nranks, f"{tag}_{os.getppid()}", group)
        arr = (ctypes.c_int32 * self.nranks)(*fds)
        st = N.nest_xsym_open(self._h, arr)
        for f in fds:   # the imported (or exported) allocations keep their own references
            os.close(f)
        if not all_ok(st):
            self.close()
            check(st if st != N.NEST_OK else N.NEST_ERR_CUDA, "nest_xsym_open (on some rank)")

    @property
    def xchunk(self) -> int:
        return int(N.nest_xsym_xchunk(self._h))

    def x_ptr(self) -> int:
        return int(N.nest_xsym_x(self._h))

    def local_x_ptr(self) -> int:
        return int(N.nest_xsym_local_x(self._h))

    def set_x(self, x_part, rank=None, stream=None):
        """Copy the first min(len, xchunk) values of x_part (a CUDA tensor) into rank r's
        slice, columns [r*xchunk, ...) (default: this rank's), stream-ordered."""
        torch = self._torch
        r = self.rank if rank is None else int(rank)
        check(N.nest_xsym_set_x(self._h, r, _dev(x_part, torch.float64, None, "x_part"), x_part.numel(),
                                _stream(stream)), "nest_xsym_set_x")

    def spmv_csr_f64(self, rowptr, colind, val, y_local=None, *, stream=None, **cfg):
        """y_local = A[local rows] @ x (global columns) on the symmetric x.  Ordering of
        the slices' writes against this call is the caller's (sync + barrier)."""
        torch = self._torch
        nrows = rowptr.numel() - 1
        nnz = val.numel()
        if y_local is None:
            y_local = torch.empty(nrows, dtype=torch.float64, device=val.device)
        d = make_desc(**cfg)
        check(N.nest_spmv_csr_f64(ctypes.byref(d), nrows, self.ncols, nnz,
                                  _dev(rowptr, torch.int64, nrows + 1, "rowptr"),
                                  _dev(colind, torch.int32, nnz, "colind"), _dev(val, torch.float64, nnz, "val"),
                                  ctypes.c_void_p(self.x_ptr()), _dev(y_local, torch.float64, nrows, "y"),
                                  _stream(stream)), "nest_spmv_csr_f64 (xsym)")
        return y_local

    def close(self):
        if self._h:
            check(N.nest_xsym_destroy(self._h), "nest_xsym_destroy")
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
