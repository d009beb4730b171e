"""The C ABI's argument checks (include/catt.h: "negative sizes and missing
pointers return CATT_EINVAL"): every compute entry point, called raw through
ctypes with a negative size or a null required pointer, returns CATT_EINVAL,
launches nothing, and leaves the device usable (an ATAX afterwards is exact)."""
import ctypes

import numpy as np
import pytest
import torch

import oracle
import seeded_inputs as si
import paper_conf_icpp_kimhlsh19_b200 as catt

pytestmark = pytest.mark.gpu

D = None  # a valid device pointer, filled in by the fixture


@pytest.fixture(scope="module", autouse=True)
def _buf():
    global D
    t = torch.zeros(1 << 20, device="cuda")
    D = ctypes.c_void_p(t.data_ptr())
    yield t


def calls():
    """(name, args with a bad size or a null pointer); D is a valid buffer."""
    N = None
    return [
        ("catt_atax", lambda: (D, D, D, D, -1, 8, N, N, N)),
        ("catt_atax", lambda: (N, D, D, D, 8, 8, N, N, N)),
        ("catt_atax", lambda: (D, D, D, D, 8, -8, N, N, N)),
        ("catt_bicg", lambda: (D, D, D, D, D, -4, 4, N, N, N)),
        ("catt_bicg", lambda: (D, N, D, D, D, 4, 4, N, N, N)),
        ("catt_mvt", lambda: (D, D, D, D, D, -4, N, N, N)),
        ("catt_mvt", lambda: (D, D, N, D, D, 4, N, N, N)),
        ("catt_gesummv", lambda: (D, D, D, D, D, -4, 1.0, 1.0, N, N)),
        ("catt_gesummv", lambda: (D, N, D, D, D, 4, 1.0, 1.0, N, N)),
        ("catt_syrk", lambda: (D, D, -4, 4, 1.0, 1.0, N, N)),
        ("catt_syrk", lambda: (N, D, 4, 4, 1.0, 1.0, N, N)),
        ("catt_syr2k", lambda: (D, D, D, 4, -4, 1.0, 1.0, N, N)),
        ("catt_syr2k", lambda: (D, N, D, 4, 4, 1.0, 1.0, N, N)),
        ("catt_gemm", lambda: (D, D, D, 4, -4, 4, 1.0, 1.0, N, N)),
        ("catt_gemm", lambda: (D, D, N, 4, 4, 4, 1.0, 1.0, N, N)),
        ("catt_corr", lambda: (D, -4, 4, D, D, D, D, N, N)),
        ("catt_corr", lambda: (N, 4, 4, D, D, D, D, N, N)),
        ("catt_kmeans_assign", lambda: (D, 8, -1, 2, D, 2, D, N, N)),
        ("catt_kmeans_assign", lambda: (D, 8, 8, 2, N, 2, D, N, N)),
        ("catt_kmeans_transpose", lambda: (D, D, -1, 2, 8, N, N)),
        ("catt_kmeans_accumulate", lambda: (D, 8, -1, 2, D, 2, D, D, N)),
        ("catt_kmeans_accumulate", lambda: (D, 8, 8, 2, D, 2, D, N, N)),
        ("catt_kmeans_finalize", lambda: (N, 2, 2, D, N, 1, N)),
        ("catt_kmeans_step", lambda: (D, 8, -1, 2, D, 2, D, D, N, N)),
        ("catt_kmeans", lambda: (D, 8, 8, 2, D, 2, D, 0, 0, D, N, N)),                # max_iter < 1
        ("catt_kmeans", lambda: (D, 8, 8, 2, D, 2, D, 4, 0, N, N, N)),                # no workspace
        ("catt_rows", lambda: (D, N, D, D, D, -4, 4, 1.0, 1.0, 0, N, N)),
        ("catt_cols", lambda: (D, D, D, -4, 4, 0, N, N)),
        ("catt_dual", lambda: (D, D, D, D, D, -4, 4, 0, 0, 0, N, N)),
        ("catt_atax_onekernel", lambda: (D, D, D, D, -1, 8, N, N, N)),
        ("catt_fill_hash", lambda: (N, 16, 1, 0, 0, N)),
        ("catt_fill_hash", lambda: (D, -16, 1, 0, 0, N)),
    ]


@pytest.mark.parametrize("i", range(len(calls())))
def test_bad_arguments_return_einval(i):
    name, args = calls()[i]
    L = catt.lib()
    torch.cuda.synchronize()
    st = getattr(L, name)(*args())
    torch.cuda.synchronize()
    assert st == catt.EINVAL, f"{name}{args()}: {L.catt_status_str(st).decode()}"


def test_device_usable_after_the_rejected_calls():
    m, n = 300, 260
    A, x = si.matrix(1, m, n), si.values(101, n)
    dev = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    tmp, y = catt.atax(dev(A), dev(x))
    tmp_o, y_o = oracle.atax(A, x)
    torch.cuda.synchronize()
    assert np.array_equal(tmp.cpu().numpy().view(np.uint32), tmp_o.view(np.uint32))
    assert np.array_equal(y.cpu().numpy().view(np.uint32), y_o.view(np.uint32))
