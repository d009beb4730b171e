"""Row-sharded ATAX (catt_atax_peer) and BICG + MVT (catt_dual_group_peer) with
the A^T partials all-reduced inside the fused kernel through peer memory
(SURVEY 8(e), 8(f) f4). This run has one GPU,
so the two ranks are two processes on cuda:0 whose buffers are mapped into
each other by CUDA IPC, exactly as on an NVLink box (where the stores cross
NVLink). Exact-dyadic inputs make every summation order bit-identical, each
rank's y must be bit-identical on every rank and every launch (both buffer
parities), equal bit for bit to the rank-order fp32 sum of the per-rank
partials that the plain fused kernel computes, and within the 1e-5 bar of the
fp64 oracle (ATAX's A^T tmp is not exact in fp32 even on dyadic inputs)."""
import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import seeded_inputs as si  # noqa: E402

TOL = 1e-5


def _relerr(got, want):
    return float(np.max(np.abs(got.astype(np.float64) - want) / np.maximum(np.abs(want), 1e-30)))


def _free_port():
    """A fresh rendezvous file for init_method="file://..." (a TCP port picked
    here could be taken by another process before the ranks bind it)."""
    import tempfile
    return os.path.join(tempfile.mkdtemp(prefix="catt_pg_"), "store")


def _init(store):
    return "file://" + store


def _problem(m, n, mode):
    A = si.matrix(si.SEED_ATAX, m, n, mode=mode)
    x = si.values(si.sub_seed(si.SEED_ATAX, 1), n, mode=mode)
    return A, x


def _rank_main(rank, world, port, m, n, steps, out_dir):
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", init_method=_init(port), rank=rank, world_size=world)
    torch.cuda.set_device(0)
    from paper_conf_icpp_kimhlsh19_b200 import dist as cdist
    import paper_conf_icpp_kimhlsh19_b200 as catt
    A, x = _problem(m, n, si.MODE_UNIFORM)
    rows = m // world
    Ag = torch.from_numpy(np.ascontiguousarray(A[rank * rows:(rank + 1) * rows])).cuda()
    xd = torch.from_numpy(x).cuda()
    peer = cdist.peer_setup(n)
    ys = []
    for _ in range(steps):
        tmp, y = cdist.atax_rowshard_peer(Ag, xd, peer)
        torch.cuda.synchronize()
        ys.append(y.cpu().numpy().copy())
    os.environ["CATT_FUSED_NO_SMALL"] = "1"          # the plain fused kernel at every shape (the peer path's tree)
    tmp_p, y_p = catt.atax(Ag, xd, k1=catt.Throttle(variant="fused"))     # this rank's partial, no exchange
    torch.cuda.synchronize()
    np.save(os.path.join(out_dir, f"y{rank}.npy"), np.stack(ys))
    np.save(os.path.join(out_dir, f"tmp{rank}.npy"), tmp.cpu().numpy())
    np.save(os.path.join(out_dir, f"part{rank}.npy"), y_p.cpu().numpy())
    np.save(os.path.join(out_dir, f"tmpp{rank}.npy"), tmp_p.cpu().numpy())
    np.save(os.path.join(out_dir, f"err{rank}.npy"), np.array([peer.timed_out()]))
    dist.barrier()
    peer.close()
    dist.destroy_process_group()


@pytest.mark.gpu
def test_atax_peer_single_rank_equals_oracle():
    import torch
    import oracle
    from paper_conf_icpp_kimhlsh19_b200 import dist as cdist
    import paper_conf_icpp_kimhlsh19_b200 as catt
    m, n = 700, 1028
    A, x = _problem(m, n, si.MODE_UNIFORM)
    t64, y64 = oracle.atax(A, x, mode=oracle.SEQ_F64)
    Ad, xd = torch.from_numpy(A).cuda(), torch.from_numpy(x).cuda()
    tmp_f, y_f = catt.atax(Ad, xd, k1=catt.Throttle(variant="fused"))
    peer = catt.Peer(1, 0, n)
    try:
        for _ in range(3):
            tmp, y = cdist.atax_rowshard_peer(Ad, xd, peer)
            torch.cuda.synchronize()
            # one rank: the same tree as the plain fused kernel, bit for bit
            assert np.array_equal(y.cpu().numpy(), y_f.cpu().numpy())
            assert np.array_equal(tmp.cpu().numpy(), tmp_f.cpu().numpy())
            assert _relerr(y.cpu().numpy(), y64) <= TOL and _relerr(tmp.cpu().numpy(), t64) <= TOL
        assert not peer.timed_out()
    finally:
        peer.close()


@pytest.mark.gpu
@pytest.mark.parametrize("world,m,n", [(2, 1024, 4096), (2, 4096, 16384), (3, 771, 260)])
def test_atax_peer_processes_share_one_gpu(tmp_path, world, m, n):
    import torch.multiprocessing as mp
    import oracle
    m -= m % world
    ctx = mp.get_context("spawn")
    port = _free_port()
    procs = [ctx.Process(target=_rank_main, args=(r, world, port, m, n, 3, str(tmp_path))) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=240)
    alive = [p for p in procs if p.is_alive()]
    for p in alive:
        p.kill()
    assert not alive, "a rank hung"
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    A, x = _problem(m, n, si.MODE_UNIFORM)
    t64, y64 = oracle.atax(A, x, mode=oracle.SEQ_F64)
    rows = m // world
    want = np.load(tmp_path / "part0.npy")
    for r in range(1, world):                            # the kernel's rank-order fp32 sum
        want = (want + np.load(tmp_path / f"part{r}.npy")).astype(np.float32)
    assert _relerr(want, y64) <= TOL
    for r in range(world):
        assert not np.load(tmp_path / f"err{r}.npy")[0]
        ys = np.load(tmp_path / f"y{r}.npy")
        for y in ys:                                     # every launch, both buffer parities
            assert np.array_equal(y, want)
        tmp = np.load(tmp_path / f"tmp{r}.npy")
        assert np.array_equal(tmp, np.load(tmp_path / f"tmpp{r}.npy"))
        assert _relerr(tmp, t64[r * rows:(r + 1) * rows]) <= TOL


# ------------------------------------------------------------------ BICG + MVT (catt_dual_group_peer)
def _bm_problem(m, n):
    A = si.matrix(si.SEED_BICG, m, n)
    B = si.matrix(si.SEED_MVT, m, n)
    p, r = si.values(si.sub_seed(si.SEED_BICG, 1), n), si.values(si.sub_seed(si.SEED_BICG, 2), m)
    y1, y2 = si.values(si.sub_seed(si.SEED_MVT, 1), n), si.values(si.sub_seed(si.SEED_MVT, 2), m)
    x1, x2 = si.values(si.sub_seed(si.SEED_MVT, 3), m), si.values(si.sub_seed(si.SEED_MVT, 4), n)
    return A, B, p, r, y1, y2, x1, x2


def _bm_group(torch, A, B, p, r, y1, y2, x1, x2, lo, hi, acc=True):
    T = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    q, s = torch.empty(hi - lo, device="cuda"), torch.empty(A.shape[1], device="cuda")
    X1, X2 = T(x1[lo:hi]), T(x2 if acc else np.zeros_like(x2))
    return [dict(A=T(A[lo:hi]), xr=T(p), xc=T(r[lo:hi]), yr=q, yc=s),
            dict(A=T(B[lo:hi]), xr=T(y1), xc=T(y2[lo:hi]), yr=X1, yc=X2, row_accumulate=True,
                 col_accumulate=acc)]


def _bm_rank_main(rank, world, port, m, n, steps, out_dir):
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", init_method=_init(port), rank=rank, world_size=world)
    torch.cuda.set_device(0)
    from paper_conf_icpp_kimhlsh19_b200 import dist as cdist
    import paper_conf_icpp_kimhlsh19_b200 as catt
    A, B, p, r, y1, y2, x1, x2 = _bm_problem(m, n)
    rows = m // world
    lo, hi = rank * rows, (rank + 1) * rows
    peer = cdist.peer_setup(2 * n)
    outs = []
    for _ in range(steps):
        g = _bm_group(torch, A, B, p, r, y1, y2, x1, x2, lo, hi)
        cdist.bicg_mvt_rowshard_peer(g, peer)
        torch.cuda.synchronize()
        outs.append([t.cpu().numpy().copy() for t in (g[0]["yr"], g[0]["yc"], g[1]["yr"], g[1]["yc"])])
    part = _bm_group(torch, A, B, p, r, y1, y2, x1, x2, lo, hi, acc=False)   # this rank's partials, no exchange
    catt.dual_group(part)
    torch.cuda.synchronize()
    for k, name in enumerate(("q", "s", "x1", "x2")):
        np.save(os.path.join(out_dir, f"{name}{rank}.npy"), np.stack([o[k] for o in outs]))
    np.save(os.path.join(out_dir, f"ps{rank}.npy"), part[0]["yc"].cpu().numpy())
    np.save(os.path.join(out_dir, f"px2{rank}.npy"), part[1]["yc"].cpu().numpy())
    np.save(os.path.join(out_dir, f"err{rank}.npy"), np.array([peer.timed_out()]))
    dist.barrier()
    peer.close()
    dist.destroy_process_group()


@pytest.mark.gpu
def test_bicg_mvt_peer_single_rank_equals_grouped_launch():
    import torch
    import paper_conf_icpp_kimhlsh19_b200 as catt
    m, n = 900, 1028
    args = _bm_problem(m, n)
    ref = _bm_group(torch, *args, 0, m)
    catt.dual_group(ref)
    peer = catt.Peer(1, 0, 2 * n)
    try:
        for _ in range(3):                                   # both buffer parities
            g = _bm_group(torch, *args, 0, m)
            catt.dual_group_peer(g, peer)
            torch.cuda.synchronize()
            for a, b in zip(g, ref):
                assert np.array_equal(a["yr"].cpu().numpy(), b["yr"].cpu().numpy())
                assert np.array_equal(a["yc"].cpu().numpy(), b["yc"].cpu().numpy())
        assert not peer.timed_out()
        with pytest.raises(catt.CattError):                  # the buffer must hold both problems' columns
            catt.dual_group_peer(_bm_group(torch, *args, 0, m), catt.Peer(1, 0, n))
    finally:
        peer.close()


@pytest.mark.gpu
@pytest.mark.parametrize("world,m,n", [(2, 4096, 4096), (3, 771, 260), (2, 1024, 16384)])
def test_bicg_mvt_peer_processes_share_one_gpu(tmp_path, world, m, n):
    """The default bench step, row-sharded: s and x2 bit-identical on every
    rank and launch, equal to the rank-order fp32 sum of the ranks' partials
    (x2: then added to its initial value), within 1e-5 of the fp64 oracle;
    q and x1 are the ranks' rows of the oracle's."""
    import torch.multiprocessing as mp
    import oracle
    m -= m % world
    ctx = mp.get_context("spawn")
    port = _free_port()
    procs = [ctx.Process(target=_bm_rank_main, args=(r, world, port, m, n, 3, str(tmp_path))) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=240)
    alive = [p for p in procs if p.is_alive()]
    for p in alive:
        p.kill()
    assert not alive, "a rank hung"
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    A, B, p, r, y1, y2, x1, x2 = _bm_problem(m, n)
    q64, s64 = oracle.bicg(A, p, r, mode=oracle.SEQ_F64)
    b1, b2 = oracle.bicg(B, y1, y2, mode=oracle.SEQ_F64)      # MVT's products (A need not be square here)
    x164, x264 = x1.astype(np.float64) + b1, x2.astype(np.float64) + b2
    ws, wx2 = np.load(tmp_path / "ps0.npy"), np.load(tmp_path / "px20.npy")
    for g in range(1, world):
        ws = (ws + np.load(tmp_path / f"ps{g}.npy")).astype(np.float32)
        wx2 = (wx2 + np.load(tmp_path / f"px2{g}.npy")).astype(np.float32)
    wx2 = (x2 + wx2).astype(np.float32)
    assert _relerr(ws, s64) <= TOL and _relerr(wx2, x264) <= TOL
    rows = m // world
    for g in range(world):
        assert not np.load(tmp_path / f"err{g}.npy")[0]
        for s_, x2_ in zip(np.load(tmp_path / f"s{g}.npy"), np.load(tmp_path / f"x2{g}.npy")):
            assert np.array_equal(s_, ws) and np.array_equal(x2_, wx2)
        for q_ in np.load(tmp_path / f"q{g}.npy"):
            assert _relerr(q_, q64[g * rows:(g + 1) * rows]) <= TOL
        for x1_ in np.load(tmp_path / f"x1{g}.npy"):
            assert _relerr(x1_, x164[g * rows:(g + 1) * rows]) <= TOL


# ------------------------------------------------------------------ unequal shards
def _uneven_rank_main(rank, world, port, rows, n, out_dir):
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", init_method=_init(port), rank=rank, world_size=world)
    torch.cuda.set_device(0)
    from paper_conf_icpp_kimhlsh19_b200 import dist as cdist
    m = sum(rows)
    A, x = _problem(m, n, si.MODE_UNIFORM)
    lo = sum(rows[:rank])
    Ag = torch.from_numpy(np.ascontiguousarray(A[lo:lo + rows[rank]])).cuda()
    peer = cdist.peer_setup(n)
    tmp, y = cdist.atax_rowshard_peer(Ag, torch.from_numpy(x).cuda(), peer)
    torch.cuda.synchronize()
    np.save(os.path.join(out_dir, f"y{rank}.npy"), y.cpu().numpy())
    np.save(os.path.join(out_dir, f"err{rank}.npy"), np.array([peer.error()]))
    dist.barrier()
    peer.close()
    dist.destroy_process_group()


def _run_uneven(tmp_path, rows, n):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    port = _free_port()
    procs = [ctx.Process(target=_uneven_rank_main, args=(r, len(rows), port, rows, n, str(tmp_path)))
             for r in range(len(rows))]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=240)
    alive = [p for p in procs if p.is_alive()]
    for p in alive:
        p.kill()
    assert not alive, "a rank hung"
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    return [int(np.load(tmp_path / f"err{r}.npy")[0]) for r in range(len(rows))]


@pytest.mark.gpu
def test_atax_peer_unequal_shards_equal_grids(tmp_path):
    """Shards of 1025 and 1024 rows launch the same grid (one CTA per SM):
    the exchange is valid and y is the oracle's on both ranks."""
    import oracle
    rows, n = [1025, 1024], 1028
    errs = _run_uneven(tmp_path, rows, n)
    assert errs == [0, 0]
    A, x = _problem(sum(rows), n, si.MODE_UNIFORM)
    _, y64 = oracle.atax(A, x, mode=oracle.SEQ_F64)
    y0, y1 = np.load(tmp_path / "y0.npy"), np.load(tmp_path / "y1.npy")
    assert np.array_equal(y0, y1) and _relerr(y0, y64) <= TOL


@pytest.mark.gpu
def test_atax_peer_grid_mismatch_is_reported_not_hung(tmp_path):
    """shards of 100 and 101 rows launch grids of 100 and 101 CTAs,
    whose chunk -> CTA maps differ. Both ranks must report the mismatch
    (catt_peer_check = 2, or 1 where a CTA had no partner) within the test's
    time limit instead of summing stale slots."""
    errs = _run_uneven(tmp_path, [100, 101], 1028)
    assert all(e in (1, 2) for e in errs) and 2 in errs, errs


# ------------------------------------------------------------------ caller-mapped (symmetric) peer memory
@pytest.mark.gpu
def test_peer_mapped_buffer_equals_grouped_launch():
    """catt_peer_create_mapped over a plain device buffer (one rank, no
    multicast alias): the per-rank store path through caller-mapped memory,
    bit-identical to the grouped launch on every launch (both parities); the
    argument checks of the mapped form."""
    import torch
    import paper_conf_icpp_kimhlsh19_b200 as catt
    m, n = 900, 1028
    args = _bm_problem(m, n)
    ref = _bm_group(torch, *args, 0, m)
    catt.dual_group(ref)
    nb = catt.Peer.nbytes(1, 2 * n)
    assert nb > 2 * 2 * n * 4
    buf = torch.zeros(nb, dtype=torch.uint8, device="cuda")
    peer = catt.Peer.mapped(1, 0, 2 * n, [buf.data_ptr()], 0, keep=buf)
    try:
        assert not peer.multicast
        for _ in range(3):
            g = _bm_group(torch, *args, 0, m)
            catt.dual_group_peer(g, peer)
            torch.cuda.synchronize()
            for a, b in zip(g, ref):
                assert np.array_equal(a["yr"].cpu().numpy(), b["yr"].cpu().numpy())
                assert np.array_equal(a["yc"].cpu().numpy(), b["yc"].cpu().numpy())
        assert not peer.timed_out()
    finally:
        peer.close()
    p2 = catt.Peer.mapped(2, 0, 2 * n, [buf.data_ptr(), buf.data_ptr()], 0, keep=buf)
    try:
        with pytest.raises(catt.CattError):                  # no IPC handles to open on a mapped peer
            p2.open(1, bytes(catt.PEER_HANDLE_BYTES))
    finally:
        p2.close()
    with pytest.raises(catt.CattError):                      # misaligned base
        catt.Peer.mapped(1, 0, 2 * n, [buf.data_ptr() + 4], 0)
    assert catt.Peer.nbytes(0, n) < 0 and catt.Peer.nbytes(1, 0) < 0


def _symm_worker(port, m, n, q):
    import torch
    import torch.distributed as dist
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", init_method=_init(port), rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        from paper_conf_icpp_kimhlsh19_b200 import dist as cdist
        import paper_conf_icpp_kimhlsh19_b200 as catt
        args = _bm_problem(m, n)
        ref = _bm_group(torch, *args, 0, m)
        catt.dual_group(ref)
        try:
            peer = cdist.peer_setup_symmetric(2 * n)
        except Exception as e:                               # symmetric memory unavailable here
            q.put(("skip", f"{type(e).__name__}: {e}"))
            return
        ok = True
        for _ in range(3):
            g = _bm_group(torch, *args, 0, m)
            catt.dual_group_peer(g, peer)
            torch.cuda.synchronize()
            for a, b in zip(g, ref):
                ok &= np.array_equal(a["yr"].cpu().numpy(), b["yr"].cpu().numpy())
                ok &= np.array_equal(a["yc"].cpu().numpy(), b["yc"].cpu().numpy())
        ok &= not peer.timed_out()
        mc = peer.multicast
        peer.close()
        q.put(("ok" if ok else "mismatch", f"multicast={mc}"))
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
def test_peer_over_torch_symmetric_memory_single_rank():
    """dist.peer_setup_symmetric (the NVSwitch form, §8(f) f4) at world 1:
    PyTorch symmetric memory as the peer buffer, the multicast alias when the
    device offers one (this one-GPU box does not: the per-rank path runs),
    results bit-identical to the grouped launch."""
    import multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    pr = ctx.Process(target=_symm_worker, args=(_free_port(), 900, 1028, q))
    pr.start()
    status, info = q.get(timeout=300)
    pr.join(timeout=60)
    if status == "skip":
        pytest.skip(f"torch symmetric memory unavailable: {info}")
    assert status == "ok" and pr.exitcode == 0, info
