"""Single-box multi-GPU scan: one process per GPU, torch.distributed for the plumbing.

Two ways to use several GPUs (PAPER.md:191-193 [§4]):

* ``mode="problems"`` -- Case 1: the G problems are split over the ranks
  (:func:`partition`), every rank scans its own problems with the single-GPU kernels.
  There is no communication at all ("Solving the Case 1 is trivial").
* ``mode="elements"`` -- Case 2, Multi-GPU Problem Scattering (Figs.
  6-7): every problem is split into rank-ordered contiguous portions.  Each rank runs
  Stage 1+2 on its portion (``shard_totals``: chunk aggregates + one total per problem),
  the totals of all ranks are exchanged with ONE all-gather of G 8-byte slots per rank
  (NCCL over NVLink/NVSwitch -- the paper's P2P writes to a master GPU and its
  MPI_Gather / MPI_Scatter, become a single collective, and every rank
  folds the totals of the ranks before it itself), then Stage 3 (``shard_scan``) scans
  the portion with that carry.  The output stays sharded like the input.

``backend="torch"`` does the exchange with ``torch.distributed.all_gather_into_tensor``
on the caller's process group; ``backend="native"`` calls the C-ABI
``scan_batch_multi`` with the group's own NCCL communicator (one library call per rank);
``backend="peer"`` (:class:`PeerComm`) makes no collective call at all: the Stage 2
kernel stores the totals straight into the later ranks' HBM over NVLink and the Stage 3
kernel waits for them on the device (the paper's P2P writes, fused
into the kernels).  All device work runs in libscanb200.so; only the sharding plan, the
one-time handle exchange and the collective call are Python.
"""
from __future__ import annotations

import ctypes

import torch
import torch.distributed as dist

from . import _lib, shard_scan, shard_totals
from ._lib import KINDS, OPS, check

__all__ = ["partition", "grouped_plan", "make_groups", "exchange_totals", "scan_multi", "NativeComm",
           "PeerComm"]


def partition(n: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous balanced split of n units: rank r owns [floor(r n / W), floor((r+1) n / W)).

    Used for problems (Case 1) and for the elements of one problem (Case 2).  Any n >= 0 and
    world >= 1 is legal; portions may be empty (the paper's Eqs. 2-3, PAPER.md:229-233,
    become "any portion length is legal").
    """
    if world < 1 or not 0 <= rank < world or n < 0:
        raise ValueError("bad partition arguments")
    return (rank * n) // world, ((rank + 1) * n) // world


def grouped_plan(G: int, N: int, world: int, V: int, rank: int) -> dict:
    """MP-PC-style grouping (PAPER.md:213-217 [§4.1.1, Fig. 8]): the W ranks form Y = W/V
    groups of V consecutive ranks; group y solves problems [floor(yG/Y), floor((y+1)G/Y))
    and, inside the group, rank v owns the contiguous portion v of each of those problems
    (the paper's "V GPUs of each PCI-e network work on G/Y problems, partitioning each
    problem into V portions of size N/V").  On NVSwitch the topology is uniform, so V only
    trades exchange fan-in against per-problem parallelism."""
    if V < 1 or world % V:
        raise ValueError("V must divide the world size")
    Y = world // V
    y, v = divmod(rank, V)
    g0, g1 = partition(G, Y, y)
    e0, e1 = partition(N, V, v)
    return {"groups": Y, "group": y, "member": v, "problems": (g0, g1), "elements": (e0, e1)}


def make_groups(V: int):
    """Create the Y = W/V sub-communicators of :func:`grouped_plan` (collective: every rank
    calls it; every rank takes part in creating every group) and return this rank's."""
    world, rank = dist.get_world_size(), dist.get_rank()
    if V < 1 or world % V:
        raise ValueError("V must divide the world size")
    mine = None
    for y in range(world // V):
        g = dist.new_group(list(range(y * V, (y + 1) * V)))
        if y == rank // V:
            mine = g
    return mine


def exchange_totals(totals: torch.Tensor, group=None) -> torch.Tensor:
    """All-gather this rank's G total slots (int64) into a rank-major [W, G] tensor."""
    world = dist.get_world_size(group)
    src = totals.contiguous().view(-1)
    if src.is_cuda and dist.get_backend(group) == "gloo":
        # gloo gathers host tensors only: stage the W*G*8 bytes through the host (plumbing
        # for CPU-backed groups, e.g. several ranks sharing one GPU in tests)
        out = torch.empty(world * src.numel(), dtype=totals.dtype)
        dist.all_gather_into_tensor(out, src.cpu(), group=group)
        return out.to(totals.device).view((world,) + tuple(totals.shape))
    out = torch.empty(world * src.numel(), dtype=totals.dtype, device=totals.device)
    dist.all_gather_into_tensor(out, src, group=group)
    return out.view((world,) + tuple(totals.shape))


class NativeComm:
    """scan_comm_t over the NCCL communicator of a torch ProcessGroupNCCL (borrowed)."""

    def __init__(self, group=None):
        pg = group if group is not None else dist.group.WORLD
        backend = pg._get_backend(torch.device("cuda", torch.cuda.current_device()))
        ptr = backend._comm_ptr()
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        h = ctypes.c_void_p(0)
        check("scan_comm_create_nccl", _lib.lib.scan_comm_create_nccl(ctypes.c_void_p(ptr), self.rank,
                                                                        self.world, ctypes.byref(h)))
        self.handle = h

    def close(self):
        if self.handle:
            check("scan_comm_destroy", _lib.lib.scan_comm_destroy(self.handle))
            self.handle = None


class PeerUnavailable(RuntimeError):
    """Raised on EVERY rank of a PeerComm set-up when any rank could not map its peers."""


class PeerComm:
    """scan_comm_t with the fused exchange over peer memory (scan_comm_create_peer).

    Setup (collective over ``group``, any backend -- gloo works): every rank creates its
    mailbox for ``max_G`` problems, the handles are all-gathered once, every rank maps the
    others'.  Afterwards ``scan_multi(..., backend="peer", comm=self)`` runs with no
    collective call.  ``PeerComm.loopback(W, max_G)`` builds W communicators inside one
    process (virtual ranks on one device, for tests)."""

    def __init__(self, max_G: int, group=None, *, rank: int | None = None, world: int | None = None,
                 _open: bool = True):
        self.rank = dist.get_rank(group) if rank is None else rank
        self.world = dist.get_world_size(group) if world is None else world
        h = ctypes.c_void_p(0)
        check("scan_comm_create_peer", _lib.lib.scan_comm_create_peer(self.rank, self.world, int(max_G),
                                                                        ctypes.byref(h)))
        self.handle = h
        self.max_G = int(max_G)
        if _open:
            blobs = [None] * self.world
            dist.all_gather_object(blobs, self.peer_handle(), group=group)
            # every rank learns whether EVERY rank mapped its peers: a rank that failed
            # (no peer access between its GPU and another's) must not leave the others to
            # spin on mailboxes it will never write -- all ranks raise the same error
            err = None
            try:
                self.open(blobs)
            except Exception as e:  # noqa: BLE001  (reported to every rank below)
                err = "%s: %s" % (type(e).__name__, e)
            errs = [None] * self.world
            dist.all_gather_object(errs, err, group=group)
            bad = [(r, e) for r, e in enumerate(errs) if e]
            if bad:
                self.close()
                raise PeerUnavailable("peer mailboxes not mapped on rank(s) %s: %s" % (
                    [r for r, _ in bad], bad[0][1]))

    def peer_handle(self) -> bytes:
        buf = ctypes.create_string_buffer(_lib.PEER_HANDLE_BYTES)
        check("scan_comm_peer_handle", _lib.lib.scan_comm_peer_handle(self.handle, buf))
        return buf.raw

    def open(self, blobs) -> None:
        if len(blobs) != self.world or any(len(b) != _lib.PEER_HANDLE_BYTES for b in blobs):
            raise ValueError("need one %d-byte handle per rank" % _lib.PEER_HANDLE_BYTES)
        allb = ctypes.create_string_buffer(b"".join(blobs), len(blobs) * _lib.PEER_HANDLE_BYTES)
        check("scan_comm_peer_open", _lib.lib.scan_comm_peer_open(self.handle, allb))

    @classmethod
    def loopback(cls, world: int, max_G: int) -> list["PeerComm"]:
        comms = [cls(max_G, rank=r, world=world, _open=False) for r in range(world)]
        blobs = [c.peer_handle() for c in comms]
        for c in comms:
            c.open(blobs)
        return comms

    def close(self):
        if self.handle:
            check("scan_comm_destroy", _lib.lib.scan_comm_destroy(self.handle))
            self.handle = None


def scan_multi(x_local: torch.Tensor, op: str = "add", kind: str = "inclusive", mode: str = "elements",
               group=None, out: torch.Tensor | None = None, backend: str = "torch",
               comm: "NativeComm | PeerComm | None" = None) -> torch.Tensor:
    """Scan this rank's share.  ``x_local`` is (G, N_local) or (N_local,).

    mode="problems": x_local holds whole problems (this rank's partition of the batch).
    mode="elements": x_local holds this rank's portion of each of the G problems.
    MP-PC grouping = mode="elements" with ``group`` = this rank's sub-communicator from
    :func:`make_groups` and x_local laid out by :func:`grouped_plan`.
    Collective in elements mode: every rank of ``group`` must call it with the same G,
    op, kind, mode and backend.
    """
    from . import scan as scan_local
    if out is None:
        out = torch.empty_like(x_local)
    if mode == "problems":
        return scan_local(x_local, op, kind, out=out)
    if mode != "elements":
        raise ValueError(mode)
    if backend in ("native", "peer"):
        N, G = (x_local.shape[0], 1) if x_local.dim() == 1 else (x_local.shape[1], x_local.shape[0])
        if comm is not None:
            c = comm
        else:
            c = NativeComm(group) if backend == "native" else PeerComm(G, group)
        from . import _dtype, _stream
        rc = _lib.lib.scan_batch_multi(x_local.data_ptr(), out.data_ptr(), N, G, OPS[op], _dtype(x_local),
                                       KINDS[kind], _stream(x_local, None), c.world, c.handle,
                                       _lib.SHARD["elements"])
        check("scan_batch_multi", rc)
        if comm is None:
            torch.cuda.current_stream().synchronize()
            if backend == "peer":         # peers may still write acks into this mailbox
                dist.barrier(group)
            c.close()
        return out
    totals = shard_totals(x_local, op)                        # Stage 1 + 2 (local)
    all_totals = exchange_totals(totals, group)               # the one exchange step
    return shard_scan(x_local, all_totals, dist.get_rank(group), dist.get_world_size(group),
                      op, kind, out=out)                      # Stage 3 (local)
