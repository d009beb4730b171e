"""Row-sharded ATAX with the A^T partials all-reduced inside the fused kernel
through peer memory (catt_atax_peer). This run has one GPU,
so the two ranks are two processes on cuda:0 whose buffers are mapped into
each other by CUDA IPC, exactly as on an NVLink box (where the stores cross
NVLink). Exact-dyadic inputs make every summation order bit-identical, each
rank's y must be bit-identical on every rank and every launch (both buffer
parities), equal bit for bit to the rank-order fp32 sum of the per-rank
partials that the plain fused kernel computes, and within the 1e-5 bar of the
fp64 oracle (ATAX's A^T tmp is not exact in fp32 even on dyadic inputs)."""
import os
import socket
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
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _problem(m, n, mode):
    A = si.matrix(si.SEED_ATAX, m, n, mode=mode)
    x = si.values(si.sub_seed(si.SEED_ATAX, 1), n, mode=mode)
    return A, x


def _rank_main(rank, world, port, m, n, steps, out_dir):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
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
