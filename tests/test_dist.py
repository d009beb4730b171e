"""Multi-process tests of the row-sharded path.

CPU, world_size 2 over gloo: the partitioning and the collective composition
of paper_conf_icpp_kimhlsh19_b200.dist with oracle-backed per-rank loops.
On exact-dyadic inputs the sharded result is bit-identical to the unsharded
oracle (every partial sum is exact, so the all-reduce order cannot matter);
on uniform inputs it is within the 1e-5 bar of the fp64 oracle.
GPU (1 device): the same functions through the CUDA kernels with a
single-rank NCCL group.
"""
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import seeded_inputs as si
from paper_conf_icpp_kimhlsh19_b200 import catt as catt_mod
from paper_conf_icpp_kimhlsh19_b200 import dist as cdist


class OracleOps:
    """Per-rank loops computed by the CPU oracle (test infrastructure). The
    accumulate forms reuse the oracle's MVT loops (init first, then the
    sequential fmaf sum), zero-padding the row shard to a square matrix."""

    @staticmethod
    def rows(A, x, y, mode, t=None, B=None, tmp=None, alpha=0.0, beta=0.0):
        An, xn = A.numpy(), x.numpy()
        m, n = An.shape
        if mode == catt_mod.ROWS_GESUMMV:
            yy, tt = oracle.gesummv(An, B.numpy(), xn, alpha, beta)
            y.copy_(torch.from_numpy(yy))
            tmp.copy_(torch.from_numpy(tt))
        elif mode == catt_mod.ROWS_ACCUM:                       # y += A x  (MVT loop 1)
            sq = np.zeros((n, n), np.float32)
            sq[:m] = An
            x1 = np.zeros(n, np.float32)
            x1[:m] = y.numpy()
            o1, _ = oracle.mvt(sq, xn, np.zeros(n, np.float32), x1, np.zeros(n, np.float32))
            y.copy_(torch.from_numpy(o1[:m].copy()))
        else:                                                   # y = A x   (BICG loop 2)
            q, _ = oracle.bicg(An, xn, np.zeros(m, np.float32))
            y.copy_(torch.from_numpy(q))
        return y

    @staticmethod
    def cols(A, v, y, accumulate, t=None):
        An, vn = A.numpy(), v.numpy()
        m, n = An.shape
        if accumulate:                                          # y += A^T v  (MVT loop 2)
            sq = np.zeros((n, n), np.float32)
            sq[:m] = An
            y2 = np.zeros(n, np.float32)
            y2[:m] = vn
            _, o2 = oracle.mvt(sq, np.zeros(n, np.float32), y2, np.zeros(n, np.float32), y.numpy())
            y.copy_(torch.from_numpy(o2))
        else:                                                   # y = A^T v   (BICG loop 1)
            _, s = oracle.bicg(An, np.zeros(n, np.float32), vn)
            y.copy_(torch.from_numpy(s))
        return y


class OracleKmeansOps:
    """Per-rank k-means steps by the oracle, writing the exact sums in the
    acc layout catt.h defines (the 128-bit two's complement of sum*2^64 as
    four 32-bit chunks, the top one signed), so that the all-reduce and the
    finalize composition of dist.kmeans_pointshard are what is tested."""

    @staticmethod
    def kmeans_accumulate(feat, ld, npoints, nf, clusters, memb, acc):
        from oracle import kmeans as okm
        cl = clusters.numpy()
        k = cl.shape[0]
        new, _ = oracle.kmeans_assign(feat.numpy(), ld, npoints, nf, cl)
        old = memb.numpy().copy()
        memb.copy_(torch.from_numpy(new))
        fe = feat.numpy()
        a = acc.numpy()
        K4 = 4 * k * nf
        for c in range(k):
            sel = np.nonzero(new == c)[0]
            a[K4 + c] += len(sel)
            for f in range(nf):
                v = okm.exact_sum(fe[f * ld + sel]) * 2 ** 64
                assert v.denominator == 1
                u = int(v) % (1 << 128)
                for l in range(4):
                    chunk = (u >> (32 * l)) & 0xFFFFFFFF
                    if l == 3 and chunk >= 1 << 31:
                        chunk -= 1 << 32
                    a[(c * nf + f) * 4 + l] += chunk
        a[K4 + k] += int(np.count_nonzero(new != old))

    @staticmethod
    def kmeans_finalize(acc, clusters, stats):
        from fractions import Fraction
        from oracle import kmeans as okm
        a = acc.numpy()
        cl = clusters.numpy()
        k, nf = cl.shape
        K4 = 4 * k * nf
        for c in range(k):
            cnt = int(a[K4 + c])
            if cnt == 0:
                continue
            for f in range(nf):
                S = sum(int(a[(c * nf + f) * 4 + l]) << (32 * l) for l in range(4))
                cl[c, f] = okm.round_f32(Fraction(S, cnt << 64))
        stats[0], stats[1], stats[2] = int(a[K4 + k]), int(a[K4 + k + 1]), int(a[K4:K4 + k].sum())
        acc.zero_()


def _free_port():
    """A fresh rendezvous file for init_method="file://..." (a TCP port picked
    here could be taken by another process before the ranks bind it)."""
    import tempfile
    return os.path.join(tempfile.mkdtemp(prefix="catt_pg_"), "store")


def _init(store):
    return "file://" + store


def _worker(rank, world, port, mode, q):
    dist.init_process_group("gloo", init_method=_init(port), rank=rank, world_size=world)
    try:
        m, n = 301, 96                                  # ragged: 151 + 150 rows
        A = si.matrix(7, m, n, mode=mode)
        x, p = si.values(8, n, mode=mode), si.values(9, n, mode=mode)
        r, y2 = si.values(10, m, mode=mode), si.values(11, m, mode=mode)
        lo, hi = cdist.row_range(m, world, rank)
        T = torch.from_numpy
        tmp_g, y = cdist.atax_rowshard(T(A[lo:hi].copy()), T(x), ops=OracleOps)
        q_g, s = cdist.bicg_rowshard(T(A[lo:hi].copy()), T(p), T(r[lo:hi].copy()), ops=OracleOps)
        sq = si.matrix(12, n, n, mode=mode)             # MVT is square
        lo2, hi2 = cdist.row_range(n, world, rank)
        x1 = si.values(13, n, mode=mode)
        x2 = T(si.values(14, n, mode=mode))
        y1 = si.values(15, n, mode=mode)
        y2s = si.values(16, n, mode=mode)
        x1_g, x2 = cdist.mvt_rowshard(T(sq[lo2:hi2].copy()), T(y1), T(y2s[lo2:hi2].copy()),
                                      T(x1[lo2:hi2].copy()), x2, ops=OracleOps)
        q.put((rank, lo, hi, tmp_g.numpy(), y.numpy(), q_g.numpy(), s.numpy(), lo2, hi2, x1_g.numpy(), x2.numpy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("mode", [si.MODE_DYADIC, si.MODE_UNIFORM])
def test_rowshard_world2_gloo(mode):
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, mode, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = sorted([q.get(timeout=180) for _ in range(world)], key=lambda t: t[0])
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    m, n = 301, 96
    A = si.matrix(7, m, n, mode=mode)
    x, p = si.values(8, n, mode=mode), si.values(9, n, mode=mode)
    r = si.values(10, m, mode=mode)
    tmp_o, y_o = oracle.atax(A, x)
    q_o, s_o = oracle.bicg(A, p, r)
    sq = si.matrix(12, n, n, mode=mode)
    x1_o, x2_o = oracle.mvt(sq, si.values(15, n, mode=mode), si.values(16, n, mode=mode),
                            si.values(13, n, mode=mode), si.values(14, n, mode=mode))
    tmp = np.concatenate([t[3] for t in res])
    q_all = np.concatenate([t[5] for t in res])
    x1 = np.concatenate([t[9] for t in res])
    assert [(t[1], t[2]) for t in res] == [(0, 151), (151, 301)]
    assert np.array_equal(tmp, tmp_o) and np.array_equal(q_all, q_o) and np.array_equal(x1, x1_o)
    for t in res:                                     # the all-reduced vectors are replicated
        assert np.array_equal(t[4], res[0][4]) and np.array_equal(t[6], res[0][6]) and np.array_equal(t[10], res[0][10])
    y, s, x2 = res[0][4], res[0][6], res[0][10]
    if mode == si.MODE_DYADIC:
        assert np.array_equal(y, y_o) and np.array_equal(s, s_o) and np.array_equal(x2, x2_o)
    else:
        _, y64 = oracle.atax(A, x, mode=oracle.SEQ_F64)
        _, s64 = oracle.bicg(A, p, r, mode=oracle.SEQ_F64)
        _, x2_64 = oracle.mvt(sq, si.values(15, n, mode=mode), si.values(16, n, mode=mode),
                              si.values(13, n, mode=mode), si.values(14, n, mode=mode), mode=oracle.SEQ_F64)
        for got, ref in ((y, y64), (s, s64), (x2, x2_64)):
            assert np.max(np.abs(got - ref) / np.abs(ref)) <= 1e-5


def _km_worker(rank, world, port, q):
    dist.init_process_group("gloo", init_method=_init(port), rank=rank, world_size=world)
    try:
        npts, nf, k = 301, 6, 3
        feat = si.values(21, nf * npts)                  # uniform, feature-major, ld = npts
        lo, hi = cdist.row_range(npts, world, rank)
        shard = np.concatenate([feat[f * npts + lo:f * npts + hi] for f in range(nf)])
        init = np.stack([feat[f * npts:f * npts + k] for f in range(nf)], axis=1)   # first k points
        cl = torch.from_numpy(init.copy())
        memb, it = cdist.kmeans_pointshard(torch.from_numpy(shard), hi - lo, hi - lo, nf, cl, max_iter=8,
                                           ops=OracleKmeansOps)
        q.put((rank, memb.numpy(), cl.numpy(), it))
    finally:
        dist.destroy_process_group()


def test_kmeans_pointshard_world2_gloo_bit_identical():
    """Integer sums: two ranks give the unsharded oracle loop's bits exactly."""
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_km_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = sorted([q.get(timeout=180) for _ in range(world)], key=lambda t: t[0])
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    from oracle import kmeans as okm
    npts, nf, k = 301, 6, 3
    feat = si.values(21, nf * npts)
    init = np.stack([feat[f * npts:f * npts + k] for f in range(nf)], axis=1)
    cl_o, memb_o, it_o, _ = okm.kmeans(feat, npts, npts, nf, init, max_iter=8)
    assert np.array_equal(np.concatenate([r[1] for r in res]), memb_o)
    for r in res:
        assert np.array_equal(r[2], cl_o) and r[3] == it_o


def test_row_range_partitions():
    for m in (0, 1, 7, 301, 65536):
        for world in (1, 2, 3, 8):
            rr = [cdist.row_range(m, world, g) for g in range(world)]
            assert rr[0][0] == 0 and rr[-1][1] == m
            assert all(rr[g][1] == rr[g + 1][0] for g in range(world - 1))
            assert max(h - l for l, h in rr) - min(h - l for l, h in rr) <= 1


@pytest.mark.gpu
def test_rowshard_single_rank_nccl():
    """The product path (CUDA kernels + NCCL) on a one-rank group."""
    dist.init_process_group("nccl", init_method=_init(_free_port()), rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        m, n = 1000, 256
        A = si.matrix(7, m, n, mode=si.MODE_DYADIC)
        x, r = si.values(8, n, mode=si.MODE_DYADIC), si.values(10, m, mode=si.MODE_DYADIC)
        tmp, y = cdist.atax_rowshard(torch.from_numpy(A).cuda(), torch.from_numpy(x).cuda(),
                                     k1=catt_mod.Throttle(variant="coop"), k2=catt_mod.Throttle(variant="coop"))
        q, s = cdist.bicg_rowshard(torch.from_numpy(A).cuda(), torch.from_numpy(x).cuda(), torch.from_numpy(r).cuda(),
                                   k1=catt_mod.Throttle(variant="staged"), k2=catt_mod.Throttle(variant="staged"))
        tmp_o, y_o = oracle.atax(A, x)
        _, y64 = oracle.atax(A, x, mode=oracle.SEQ_F64)
        q_o, s_o = oracle.bicg(A, x, r)
        torch.cuda.synchronize()
        # tmp is exact (dyadic); y multiplies by the derived tmp, so partial sums
        # exceed 2^24 ulps and the coop order may differ: fp64 bar
        assert np.array_equal(tmp.cpu().numpy(), tmp_o)
        assert np.max(np.abs(y.cpu().numpy() - y64) / np.abs(y64)) <= 1e-5
        assert np.array_equal(q.cpu().numpy(), q_o) and np.array_equal(s.cpu().numpy(), s_o)
    finally:
        dist.destroy_process_group()


class _FakePeer:
    """Stands in for catt.Peer on CPU: records which handles were opened."""

    def __init__(self, world, rank, n):
        self.world, self.rank, self.n = world, rank, n
        self.handle = bytes([rank]) * catt_mod.PEER_HANDLE_BYTES
        self.opened = {}

    def open(self, r, h):
        assert r not in self.opened
        self.opened[r] = h


def _peer_worker(rank, world, port, q):
    dist.init_process_group("gloo", init_method=_init(port), rank=rank, world_size=world)
    try:
        orig = catt_mod.Peer
        catt_mod.Peer = _FakePeer
        try:
            p = cdist.peer_setup(4096)
        finally:
            catt_mod.Peer = orig
        q.put((rank, p.world, p.rank, sorted(p.opened), {r: h[0] for r, h in p.opened.items()}))
    finally:
        dist.destroy_process_group()


def test_peer_setup_exchanges_handles_world3_gloo():
    """Host side of the fused peer all-reduce (f4): every rank creates one
    peer object and opens every other rank's IPC handle exactly once (its own
    never), over a gloo group of 3 processes."""
    world, port = 3, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_peer_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert all(p.exitcode == 0 for p in procs)
    for rank, w, r, opened, first_bytes in res:
        assert (w, r) == (world, rank)
        assert opened == [x for x in range(world) if x != rank]
        assert all(first_bytes[x] == x for x in opened)          # the handle of rank x came from rank x


def _cuda_worker(rank, world, port, mode, q):
    """The row-sharded and point-sharded paths through the CUDA kernels
    (CudaOps, libcatt.so) in world processes that share cuda:0, with gloo
    collectives on the CUDA tensors (NCCL needs one GPU per rank; this run
    has one GPU)."""
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method=_init(port), rank=rank, world_size=world)
    try:
        C = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
        H = lambda t: (torch.cuda.synchronize(), t.cpu().numpy())[1]
        m, n = 4099, 1024                               # ragged: 2050 + 2049 rows, several CTAs per rank
        A = si.matrix(7, m, n, mode=mode)
        x, p = si.values(8, n, mode=mode), si.values(9, n, mode=mode)
        r = si.values(10, m, mode=mode)
        lo, hi = cdist.row_range(m, world, rank)
        tmp_g, y = cdist.atax_rowshard(C(A[lo:hi]), C(x))
        q_g, s = cdist.bicg_rowshard(C(A[lo:hi]), C(p), C(r[lo:hi]))
        sq = si.matrix(12, n, n, mode=mode)
        lo2, hi2 = cdist.row_range(n, world, rank)
        x1, x2 = si.values(13, n, mode=mode), C(si.values(14, n, mode=mode))
        y1, y2s = si.values(15, n, mode=mode), si.values(16, n, mode=mode)
        x1_g, x2 = cdist.mvt_rowshard(C(sq[lo2:hi2]), C(y1), C(y2s[lo2:hi2]), C(x1[lo2:hi2]), x2)
        ng = 1027                                        # GESUMMV is square: 514 + 513 rows
        Ag, Bg, xg = si.matrix(18, ng, ng, mode=mode), si.matrix(17, ng, ng, mode=mode), si.values(19, ng, mode=mode)
        lo4, hi4 = cdist.row_range(ng, world, rank)
        yg, tg = cdist.gesummv_rowshard(C(Ag[lo4:hi4]), C(Bg[lo4:hi4]), C(xg), 1.5, 1.25)
        npts, nf, k = 3001, 6, 3                        # k-means, point-sharded, exact sums
        feat = si.values(21, nf * npts)
        lo3, hi3 = cdist.row_range(npts, world, rank)
        shard = np.concatenate([feat[f * npts + lo3:f * npts + hi3] for f in range(nf)])
        init = np.stack([feat[f * npts:f * npts + k] for f in range(nf)], axis=1)
        cl = C(init)
        memb, it = cdist.kmeans_pointshard(C(shard), hi3 - lo3, hi3 - lo3, nf, cl, max_iter=8)
        q.put((rank, lo, hi, H(tmp_g), H(y), H(q_g), H(s), H(x1_g), H(x2), H(yg), H(tg), H(memb), H(cl), int(it)))
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.parametrize("mode", [si.MODE_DYADIC, si.MODE_UNIFORM])
def test_rowshard_world2_cuda_kernels_gloo(mode):
    """§8(e) at world 2 through the CUDA kernels: ATAX / BICG / MVT / GESUMMV
    row-sharded and KMEANS point-sharded, every rank's outputs against the
    oracle: row outputs bit-exact; the all-reduced column outputs bit-exact to
    the per-shard oracle partials summed in fp32 (and, uniform inputs, within
    1e-5 of the unsharded fp64 oracle); k-means bit-identical to the
    unsharded oracle loop."""
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_cuda_worker, args=(r, world, port, mode, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = sorted([q.get(timeout=300) for _ in range(world)], key=lambda t: t[0])
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    m, n = 4099, 1024
    A = si.matrix(7, m, n, mode=mode)
    x, p = si.values(8, n, mode=mode), si.values(9, n, mode=mode)
    r = si.values(10, m, mode=mode)
    sq = si.matrix(12, n, n, mode=mode)
    mv = (sq, si.values(15, n, mode=mode), si.values(16, n, mode=mode), si.values(13, n, mode=mode),
          si.values(14, n, mode=mode))
    ng = 1027
    tmp_o, y_o = oracle.atax(A, x)
    q_o, s_o = oracle.bicg(A, p, r)
    x1_o, x2_o = oracle.mvt(*mv)
    yg_o, tg_o = oracle.gesummv(si.matrix(18, ng, ng, mode=mode), si.matrix(17, ng, ng, mode=mode),
                                si.values(19, ng, mode=mode), 1.5, 1.25)
    cat = lambda i: np.concatenate([t[i] for t in res])
    # row outputs: each rank's rows, sequential per row in every variant the default plan picks
    assert np.array_equal(cat(3), tmp_o) and np.array_equal(cat(9), yg_o) and np.array_equal(cat(10), tg_o)
    assert np.array_equal(cat(5), q_o) and np.array_equal(cat(7), x1_o)
    for t in res:                                     # the all-reduced outputs are replicated
        for i in (4, 6, 8):
            assert np.array_equal(t[i], res[0][i])
    # the all-reduced outputs: each rank's partial is its shard's sequential
    # column loop (the oracle on the shard), and the world-2 SUM is one fp32
    # add of the two partials: bit-exact in both modes
    T = torch.from_numpy
    parts = {"y": [], "s": [], "x2": []}
    for g in range(2):
        lo, hi = cdist.row_range(m, 2, g)
        tmp_g, _ = oracle.atax(A[lo:hi], x)
        parts["y"].append(OracleOps.cols(T(A[lo:hi].copy()), T(tmp_g), torch.empty(n), False).numpy())
        parts["s"].append(OracleOps.cols(T(A[lo:hi].copy()), T(r[lo:hi].copy()), torch.empty(n), False).numpy())
        lo2, hi2 = cdist.row_range(n, 2, g)
        x2_init = mv[4].copy() if g == 0 else np.zeros(n, np.float32)
        parts["x2"].append(OracleOps.cols(T(sq[lo2:hi2].copy()), T(mv[2][lo2:hi2].copy()), T(x2_init), g == 0).numpy())
    for key, i in (("y", 4), ("s", 6), ("x2", 8)):
        want = (parts[key][0] + parts[key][1]).astype(np.float32)
        assert np.array_equal(res[0][i], want), key
    if mode == si.MODE_UNIFORM:                       # and within the 1e-5 bar of fp64
        _, y64 = oracle.atax(A, x, mode=oracle.SEQ_F64)
        _, s64 = oracle.bicg(A, p, r, mode=oracle.SEQ_F64)
        _, x2_64 = oracle.mvt(*mv, mode=oracle.SEQ_F64)
        for got, ref in ((res[0][4], y64), (res[0][6], s64), (res[0][8], x2_64)):
            assert np.max(np.abs(got - ref) / np.abs(ref)) <= 1e-5
    from oracle import kmeans as okm
    npts, nf, k = 3001, 6, 3
    feat = si.values(21, nf * npts)
    init = np.stack([feat[f * npts:f * npts + k] for f in range(nf)], axis=1)
    cl_o, memb_o, it_o, _ = okm.kmeans(feat, npts, npts, nf, init, max_iter=8)
    assert np.array_equal(cat(11), memb_o)
    for t in res:
        assert np.array_equal(t[12], cl_o) and t[13] == it_o
