"""Row-sharded multi-GPU ATAX / BICG / MVT / GESUMMV.

One process per GPU (torch.distributed, NCCL over NVLink/NVSwitch). Rows of A
are split across ranks; every rank runs the CATT-throttled loops on its own
rows through the C ABI, and the A^T partial sums are added with one
all_reduce(SUM) -- the only exchange these loops have:

    ATAX   tmp_g = A_g x (local),      y = sum_g A_g^T tmp_g        (all-reduce)
    BICG   q_g   = A_g p (local),      s = sum_g A_g^T r_g          (all-reduce)
    MVT    x1_g += A_g y1 (local),     x2 = x2 + sum_g A_g^T y2_g   (all-reduce;
           only rank 0 adds the initial x2, so the sum carries it once)
    GESUMMV y_g = alpha A_g x + beta B_g x (local, no collective)
    KMEANS points sharded; per iteration the exact centroid sums (int64 limbs,
           counts, delta) are all-reduced, then every rank finalizes the
           same centres. Integer sums: the result is
           bit-identical at any world size.

The per-rank loop calls are injected (`ops`), so the partitioning and the
collective composition can be tested on CPU over gloo with any loop
implementation; the default ops are the CUDA kernels (catt.rows / catt.cols).
"""
from __future__ import annotations

from typing import Callable, Optional, Tuple

from . import catt


def row_range(m: int, world: int, rank: int) -> Tuple[int, int]:
    """Contiguous, balanced row block [lo, hi) of rank `rank` (first m % world ranks get one more)."""
    base, extra = divmod(m, world)
    lo = rank * base + min(rank, extra)
    return lo, lo + base + (1 if rank < extra else 0)


class CudaOps:
    """Per-rank loops on the local GPU (the product path)."""

    @staticmethod
    def rows(A, x, y, mode, t=None, B=None, tmp=None, alpha=0.0, beta=0.0):
        return catt.rows(A, x, y, mode, B=B, tmp=tmp, alpha=alpha, beta=beta, t=t)

    @staticmethod
    def cols(A, v, y, accumulate, t=None):
        return catt.cols(A, v, y, accumulate, t=t)

    @staticmethod
    def kmeans_accumulate(feat, ld, npoints, nf, clusters, memb, acc):
        catt.kmeans_accumulate(feat, ld, npoints, nf, clusters, memb, acc)

    @staticmethod
    def kmeans_finalize(acc, clusters, stats):
        catt.kmeans_finalize(acc, clusters, stats, zero_acc=True)


def _reduce(t, group):
    import torch.distributed as dist
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return t


def _rank(group):
    import torch.distributed as dist
    return dist.get_rank(group) if dist.is_initialized() else 0


def atax_rowshard(A_g, x, tmp_g=None, y=None, k1=None, k2=None, group=None, ops=CudaOps):
    """tmp_g = A_g x; y = sum over ranks of A_g^T tmp_g."""
    import torch
    m, n = A_g.shape
    tmp_g = torch.empty(m, dtype=A_g.dtype, device=A_g.device) if tmp_g is None else tmp_g
    y = torch.empty(n, dtype=A_g.dtype, device=A_g.device) if y is None else y
    ops.rows(A_g, x, tmp_g, catt.ROWS_STORE, k1)
    ops.cols(A_g, tmp_g, y, False, k2)
    _reduce(y, group)
    return tmp_g, y


def peer_setup(n, group=None):
    """This rank's catt.Peer for n columns: its CUDA IPC
    handle goes to every rank of the group (all_gather_object) and the other
    ranks' buffers are opened. One per (group, n); reuse it for every step."""
    import torch.distributed as dist
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = _rank(group)
    peer = catt.Peer(world, rank, n)
    if world > 1:
        handles = [None] * world
        dist.all_gather_object(handles, (rank, peer.handle), group=group)
        for r, h in handles:
            if r != rank:
                peer.open(r, h)
    return peer


def peer_setup_symmetric(n, group=None):
    """This rank's catt.Peer over PyTorch symmetric memory (SURVEY 8(f) f4,
    the NVSwitch form): every rank's buffer mapped into every process, and,
    where the device and driver support NVLS multicast, a multicast alias so
    the in-kernel all-reduce stores each partial once (multimem.st) instead
    of once per rank. Falls back to per-rank stores through the mapped
    buffers when there is no multicast (peer.multicast tells which). Needs an
    initialised process group (NCCL) with one GPU per rank."""
    import torch
    import torch.distributed as dist
    import torch.distributed._symmetric_memory as symm
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    nb = catt.Peer.nbytes(world, n)
    buf = symm.empty(nb, dtype=torch.uint8, device=torch.device("cuda", torch.cuda.current_device()))
    buf.zero_()
    h = symm.rendezvous(buf, group if group is not None else dist.group.WORLD)
    torch.cuda.synchronize()
    h.barrier()
    try:                                  # 0 where the device or driver offers no NVLS multicast
        mc = int(h.multicast_ptr or 0)
    except (RuntimeError, AttributeError):
        mc = 0
    return catt.Peer.mapped(world, rank, n, [int(p) for p in h.buffer_ptrs], mc, keep=(buf, h))


def atax_rowshard_peer(A_g, x, peer, tmp_g=None, y=None):
    """tmp_g = A_g x; y = sum over ranks of A_g^T tmp_g, with the sum done
    inside the fused kernel through peer memory (no NCCL call): one launch
    per step on every rank, y bit-identical on all ranks."""
    return catt.atax_peer(A_g, x, peer, tmp_g, y)


def bicg_mvt_rowshard_peer(problems, peer):
    """The grouped single-read step (catt_dual_group_peer) on this rank's rows
    of every problem: row outputs local, column outputs (BICG's s, MVT's x2)
    summed over ranks inside the kernel through peer memory (no NCCL call),
    bit-identical on all ranks. `peer` from peer_setup(n * len(problems))."""
    catt.dual_group_peer(problems, peer)
    return problems


def bicg_rowshard(A_g, p, r_g, q_g=None, s=None, k1=None, k2=None, group=None, ops=CudaOps):
    """s = sum over ranks of A_g^T r_g (k1); q_g = A_g p (k2)."""
    import torch
    m, n = A_g.shape
    q_g = torch.empty(m, dtype=A_g.dtype, device=A_g.device) if q_g is None else q_g
    s = torch.empty(n, dtype=A_g.dtype, device=A_g.device) if s is None else s
    ops.cols(A_g, r_g, s, False, k1)
    ops.rows(A_g, p, q_g, catt.ROWS_STORE, k2)
    _reduce(s, group)
    return q_g, s


def mvt_rowshard(A_g, y1, y2_g, x1_g, x2, k1=None, k2=None, group=None, ops=CudaOps):
    """x1_g += A_g y1 (local rows); x2 = x2 + sum over ranks of A_g^T y2_g.
    A_g is the rank's rows of the square A; x2 is replicated, updated in place."""
    ops.rows(A_g, y1, x1_g, catt.ROWS_ACCUM, k1)
    ops.cols(A_g, y2_g, x2, _rank(group) == 0, k2)   # only rank 0 carries the initial x2
    _reduce(x2, group)
    return x1_g, x2


def gesummv_rowshard(A_g, B_g, x, alpha, beta, y_g=None, tmp_g=None, t=None, ops=CudaOps):
    """y_g = alpha A_g x + beta B_g x, tmp_g = A_g x: fully local, no collective."""
    import torch
    m = A_g.shape[0]
    y_g = torch.empty(m, dtype=A_g.dtype, device=A_g.device) if y_g is None else y_g
    tmp_g = torch.empty(m, dtype=A_g.dtype, device=A_g.device) if tmp_g is None else tmp_g
    ops.rows(A_g, x, y_g, catt.ROWS_GESUMMV, t, B=B_g, tmp=tmp_g, alpha=alpha, beta=beta)
    return y_g, tmp_g


def kmeans_pointshard(feat_g, ld_g, npoints_g, nf, clusters, memb_g=None, max_iter=500, max_changes=0, group=None,
                      ops=CudaOps):
    """k-means over points sharded across ranks. feat_g is this rank's points,
    feature-major (feat_g[f*ld_g + p]); clusters (k x nf) is replicated and
    updated in place. Per iteration: assignment + exact sums on the local
    points, all_reduce(SUM) of the int64 sums/counts/delta (the iteration's
    one exchange), then every rank rounds the same means. Returns
    (memb_g, iterations)."""
    import torch
    k = clusters.shape[0]
    acc = torch.zeros(catt.kmeans_acc_words(k, nf), dtype=torch.int64, device=clusters.device)
    stats = torch.zeros(3, dtype=torch.int64, device=clusters.device)
    if memb_g is None:
        memb_g = torch.empty(npoints_g, dtype=torch.int32, device=clusters.device)
    memb_g.fill_(-1)
    it = 0
    while it < max_iter:
        ops.kmeans_accumulate(feat_g, ld_g, npoints_g, nf, clusters, memb_g, acc)
        _reduce(acc, group)
        ops.kmeans_finalize(acc, clusters, stats)
        it += 1
        if int(stats[0].item()) <= max_changes:            # global delta (all-reduced)
            break
    return memb_g, it
