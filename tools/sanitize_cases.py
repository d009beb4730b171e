"""Small launches of every synchronisation mechanism in libcatt.so, one case
per process, for compute-sanitizer (racecheck / synccheck / memcheck /
initcheck). Run:  compute-sanitizer --tool racecheck python tools/sanitize_cases.py <case>

Mechanisms:
  gate_sem      warp gate: shared-memory semaphore (atomicSub/atomicAdd + nanosleep)
  gate_barrier  warp gate: Fig 4 groups separated by __syncthreads (ragged rows)
  cta_counter   CTA cap: per-SM counter in global memory (spin on %smid slot)
  smem_pad      CTA cap: Fig 5 dynamic shared-memory pad
  staged        TMA rows/cols rings (full/empty mbarriers)
  coop          COOP rows (warp tree) / cols (cluster DSMEM)
  fused         catt_dual / catt_dual_group (bulk-copy ring, arrival counters, grid barrier)
  fused_graph   the fused grouped kernel captured in a CUDA graph (self-resetting barrier)
  onekernel     both ATAX loops in one cooperative kernel (grid barrier)
  kmeans        assign (literal gated, staged TMA ring, coop) + transpose
  km_iter       km_accumulate + finalize + the one-launch loop
  tiles         SYRK / SYR2K / GEMM / CORR tiled kernels
  tiles2        the two-CTA-per-SM tile kernel T2 (prep transpose, TMA ring with
                full/empty mbarriers, 64- and 48-row tiles, ragged n and m, tri)
  peer          one rank of the peer-memory all-reduce (launch 2 under torchrun)
Every case checks its result against the CPU oracle so a silent corruption
under the sanitizer is also caught.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402
import seeded_inputs as si  # noqa: E402

D = si.MODE_DYADIC


def T(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def eq(got, want, what):
    got = got.cpu().numpy() if isinstance(got, torch.Tensor) else got
    assert np.array_equal(got, want), what


def rows_case(t, m=700, n=96):
    A, x = si.matrix(1, m, n, D), si.values(101, n, mode=D)
    tmp, y = catt.atax(T(A), T(x), k1=t)
    t_o, y_o = oracle.atax(A, x)
    eq(tmp, t_o, "tmp")
    eq(y, y_o, "y")


def case_gate_sem():
    rows_case(catt.Throttle(active_warps=2))
    rows_case(catt.Throttle(active_warps=3, cta_threads=192), m=333)


def case_gate_barrier():
    rows_case(catt.Throttle(active_warps=4, gate=catt.GATE_BARRIER), m=700)
    rows_case(catt.Throttle(active_warps=1, gate=catt.GATE_BARRIER, cta_threads=128), m=130)


def case_cta_counter():
    # more CTAs than 148 SMs x cap so the counter actually blocks
    rows_case(catt.Throttle(active_ctas=1, cta_threads=64), m=148 * 64 * 3 + 17, n=40)
    rows_case(catt.Throttle(active_warps=1, active_ctas=2, cta_threads=128), m=148 * 128 * 3, n=40)


def case_smem_pad():
    rows_case(catt.Throttle(active_ctas=2, cap=catt.CAP_SMEM_PAD, carveout_kb=64), m=148 * 256 * 3, n=40)


def case_staged():
    rows_case(catt.Throttle(variant="staged"), m=1000, n=200)
    A, p, r = si.matrix(2, 777, 300, D), si.values(102, 300, mode=D), si.values(202, 777, mode=D)
    q, s = catt.bicg(T(A), T(p), T(r), k1=catt.Throttle(variant="staged"), k2=catt.Throttle(variant="staged"))
    qo, so = oracle.bicg(A, p, r)
    eq(q, qo, "q")
    eq(s, so, "s")


def case_coop():
    A, p, r = si.matrix(2, 777, 300, D), si.values(102, 300, mode=D), si.values(202, 777, mode=D)
    q, s = catt.bicg(T(A), T(p), T(r), k1=catt.Throttle(variant="coop"), k2=catt.Throttle(variant="coop"))
    qo, so = oracle.bicg(A, p, r)
    eq(q, qo, "q")
    eq(s, so, "s")
    B, x = si.matrix(5, 300, 300, D), si.values(105, 300, mode=D)
    y, tmp = catt.gesummv(T(A[:300]), T(B), T(x), 1.5, 1.25, t=catt.Throttle(variant="coop"))
    yo, to = oracle.gesummv(A[:300], B, x, 1.5, 1.25)
    eq(y, yo, "gesummv y")


def _dual_problems(nb):
    Ab, Am = si.matrix(2, nb, nb, D), si.matrix(3, nb, nb, D)
    pv, rv, y1, y2 = (si.values(s, nb, mode=D) for s in (102, 202, 103, 203))
    x1, x2 = si.values(104, nb, mode=D), si.values(204, nb, mode=D)
    want = oracle.bicg(Ab, pv, rv) + oracle.mvt(Am, y1, y2, x1, x2)
    qd, sd = torch.empty(nb, device="cuda"), torch.empty(nb, device="cuda")
    x1d, x2d = T(x1), T(x2)
    probs = [dict(A=T(Ab), xr=T(pv), xc=T(rv), yr=qd, yc=sd),
             dict(A=T(Am), xr=T(y1), xc=T(y2), yr=x1d, yc=x2d, row_accumulate=True, col_accumulate=True)]
    return probs, (qd, sd, x1d, x2d), want, (x1, x2)


def case_fused():
    probs, outs, want, _ = _dual_problems(384)
    catt.dual_group(probs)
    for g, w_, nm in zip(outs, want, "q s x1 x2".split()):
        eq(g, w_, nm)
    A, x = si.matrix(1, 500, 260, D), si.values(101, 260, mode=D)
    os.environ["CATT_FUSED_NO_SMALL"] = "1"
    tmp, y = catt.atax(T(A), T(x), k1=catt.Throttle(variant="fused"))       # grid barrier (dependent)
    t_o, y_o = oracle.atax(A, x, mode=oracle.SEQ_F64)
    assert np.max(np.abs(y.cpu().numpy() - y_o) / y_o) < 1e-5
    os.environ.pop("CATT_FUSED_NO_SMALL")
    tmp, y = catt.atax(T(A[:200, :256]), T(x[:256]), k1=catt.Throttle(variant="fused"))   # small cluster form
    t_o, y_o = oracle.atax(A[:200, :256], x[:256], mode=oracle.SEQ_F64)
    assert np.max(np.abs(y.cpu().numpy() - y_o) / y_o) < 1e-5


def case_fused_graph():
    probs, outs, want, (x1, x2) = _dual_problems(384)
    s = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        catt.dual_group(probs)               # warm-up outside capture
    torch.cuda.synchronize()
    outs[2].copy_(T(x1))
    outs[3].copy_(T(x2))
    with torch.cuda.graph(g, stream=s):
        catt.dual_group(probs)
    for _ in range(2):
        outs[2].copy_(T(x1))
        outs[3].copy_(T(x2))
        g.replay()
        torch.cuda.synchronize()
        for gt, w_, nm in zip(outs, want, "q s x1 x2".split()):
            eq(gt, w_, nm)


def case_onekernel():
    A, x = si.matrix(1, 600, 200, D), si.values(101, 200, mode=D)
    tmp, y = catt.atax_onekernel(T(A), T(x), k1=catt.Throttle(active_warps=2), k2=catt.Throttle(active_warps=4))
    t_o, y_o = oracle.atax(A, x)
    eq(tmp, t_o, "tmp")
    eq(y, y_o, "y")


def case_kmeans():
    npts, nf, k, ld = 3001, 34, 5, 3004
    feat = si.values(4, nf * ld)
    cl = feat.reshape(nf, ld)[:, :k].T.copy()
    want, _ = oracle.kmeans_assign(feat, ld, npts, nf, cl)
    for t in (catt.Throttle(active_warps=2, active_ctas=1), catt.Throttle(variant="staged"),
              catt.Throttle(variant="coop"), catt.Throttle(variant="regs")):
        memb = catt.kmeans_assign(T(feat), ld, npts, nf, T(cl), t=t)
        eq(memb, want, f"membership {t}")
    pm = feat.reshape(nf, ld)[:, :npts].T.copy()          # point-major
    for t in (catt.Throttle(active_warps=4), catt.Throttle(variant="coop")):
        out = torch.zeros(nf * ld, device="cuda")
        catt.kmeans_transpose(T(pm), npts, nf, out, ld, t=t)
        eq(out.view(nf, ld)[:, :npts], pm.T, f"transpose {t}")


def case_km_iter():
    from oracle import kmeans as okm
    npts, nf, k, ld = 3001, 34, 5, 3003
    feat = si.values(4, nf * ld)
    cl = feat.reshape(nf, ld)[:, :k].T.copy()
    memb_o, _ = oracle.kmeans_assign(feat, ld, npts, nf, cl)
    C = T(cl)
    acc = torch.zeros(catt.kmeans_acc_words(k, nf), dtype=torch.int64, device="cuda")
    mk = torch.full((npts,), -1, dtype=torch.int32, device="cuda")
    catt.kmeans_accumulate(T(feat), ld, npts, nf, C, mk, acc)
    catt.kmeans_finalize(acc, C)
    cl_o, _ = okm.update(feat, ld, npts, nf, memb_o, cl)
    eq(C, cl_o, "centres")
    C2 = T(cl)
    res = catt.kmeans(T(feat), ld, npts, nf, C2, max_iter=3)
    want = okm.kmeans(feat, ld, npts, nf, cl, max_iter=3)
    eq(C2, want[0], "kmeans loop centres")


def case_tiles():
    n, m = 160, 72
    A, B = si.matrix(6, n, m, D), si.matrix(8, n, m, D)
    C0 = si.matrix(9, n, n, D)
    C = T(C0)
    catt.syrk(T(A), C, 1.5, 1.25, t=catt.Throttle(variant="staged"))
    eq(C, oracle.syrk(A, C0, 1.5, 1.25), "syrk")
    C = T(C0)
    catt.syr2k(T(A), T(B), C, 1.5, 1.25, t=catt.Throttle(variant="staged"))
    eq(C, oracle.syr2k(A, B, C0, 1.5, 1.25), "syr2k")
    G = si.matrix(10, m, n, D)
    Cg = si.matrix(11, n, n, D)
    C = T(Cg)
    catt.gemm(T(A), T(G), C, 1.5, 1.25, t=catt.Throttle(variant="staged"))
    eq(C, oracle.gemm(A, G, Cg, 1.5, 1.25), "gemm")
    data = si.matrix(12, 130, 70)
    sym = catt.corr(T(data), t=catt.Throttle(variant="staged"))[0]
    eq(sym, oracle.corr(data)[0], "corr")


def case_tiles2():
    n, m = 1601, 40                                   # the mixed 56-row tile, ragged edge and last stage
    A, B = si.matrix(6, n, m, D), si.matrix(8, n, m, D)
    C0 = si.matrix(9, n, n, D)
    C = T(C0)
    catt.syrk(T(A), C, 1.5, 1.25, t=catt.Throttle(variant="staged"))
    eq(C, oracle.syrk(A, C0, 1.5, 1.25), "syrk T2 (mixed tile)")
    n1 = 1001                                         # SYR2K through the mixed tile: 7 warps in the last CTA
    C0 = si.matrix(9, n1, n1, D)
    C = T(C0)
    catt.syr2k(T(A[:n1]), T(B[:n1]), C, 1.5, 1.25, t=catt.Throttle(variant="staged"))
    eq(C, oracle.syr2k(A[:n1], B[:n1], C0, 1.5, 1.25), "syr2k T2 (mixed tile)")
    n3, m3 = 2200, 8                                  # more than one wave: the uniform 64-row tile
    A3 = si.matrix(7, n3, m3, D)
    C0 = si.matrix(9, n3, n3, D)
    C = T(C0)
    catt.syrk(T(A3), C, 1.5, 1.25, t=catt.Throttle(variant="staged"))
    eq(C, oracle.syrk(A3, C0, 1.5, 1.25), "syrk T2 (uniform tile)")
    n2 = 300
    C0 = si.matrix(9, n2, n2, D)
    C = T(C0)
    catt.syr2k(T(A[:n2]), T(B[:n2]), C, 1.5, 1.25, t=catt.Throttle(variant="staged"))
    eq(C, oracle.syr2k(A[:n2], B[:n2], C0, 1.5, 1.25), "syr2k T2")
    data = si.matrix(12, 24, n)                       # n columns: the upper tiles through T2 (transposed form)
    sym = catt.corr(T(data), t=catt.Throttle(variant="staged"))[0]
    eq(sym, oracle.corr(data)[0], "corr T2")
    data = si.matrix(13, 300, 1604)                   # m % 4 == 0: strip statistics (TMA boxes) + T2 on the data
    sym = catt.corr(T(data), t=catt.Throttle(variant="staged"))[0]
    eq(sym, oracle.corr(data)[0], "corr direct")


def case_peer():
    import torch.distributed as dist
    from paper_conf_icpp_kimhlsh19_b200 import dist as cdist
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    torch.cuda.set_device(0)
    m, n = 256 * world, 1028
    A, x = si.matrix(si.SEED_ATAX, m, n, D), si.values(si.sub_seed(si.SEED_ATAX, 1), n, mode=D)
    rows = m // world
    peer = cdist.peer_setup(n)
    Ag = T(A[rank * rows:(rank + 1) * rows])
    for _ in range(3):
        tmp, y = cdist.atax_rowshard_peer(Ag, T(x), peer)
        torch.cuda.synchronize()
    assert not peer.timed_out()
    probs, outs, want, _ = _dual_problems(256)
    dist.barrier()
    peer.close()
    peer2 = cdist.peer_setup(2 * 256)
    cdist.bicg_mvt_rowshard_peer(probs, peer2)
    torch.cuda.synchronize()
    assert not peer2.timed_out()
    dist.barrier()
    peer2.close()
    dist.destroy_process_group()


CASES = {k[5:]: v for k, v in globals().items() if k.startswith("case_")}

if __name__ == "__main__":
    names = sys.argv[1:] or sorted(c for c in CASES if c != "peer")   # peer runs under torchrun
    for nm in names:
        CASES[nm]()
        torch.cuda.synchronize()
        print(f"case {nm}: ok", flush=True)
