"""tiles_per_cta (consecutive workgroup-level tiles per CTA, a B200 scheduling knob) is
launch-time only: y must be BITWISE identical for every value — same tiles, same
association (Q10) — in both strategies, with the power-step epilogue, BCCOO+
slices, the seg_row map, and the forced hand-off path; and integer data stays exact."""
import numpy as np
import pytest

import synth
from oracle import encode as E, ref

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_yanlzz14_b200  # noqa: F401


def _bits(y):
    return y.view(np.uint32 if y.dtype == np.float32 else np.uint64)


CASES = [
    ("c1", dict(T=4, C=64)),
    ("c3-ship", dict(h=2, w=2, T=8, C=128)),
    ("c4", dict(T=8, C=64)),
    ("c4", dict(T=8, C=128, S=3)),
    ("c4", dict(T=16, C=64, empty_mode=E.EMPTY_MAP, col_mode=E.COL_DELTA)),
]


@pytest.mark.parametrize("name,p", CASES)
@pytest.mark.parametrize("rc", [0, 1])
@pytest.mark.parametrize("flags", [0, 32])
def test_bitwise_across_tiles_per_cta(name, p, rc, flags):
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    csr = synth.config_matrix(name)
    x = torch.from_numpy(synth.make_x(csr.n, csr.val.dtype, "uniform", 2)).cuda()
    A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=0, rc=rc, flags=flags, tpc=1, **p)
    try:
        y1 = A.spmv(x).cpu().numpy()
        y_ref, bound = ref.spmv(csr.row_ptr, csr.col, csr.val, x.cpu().numpy())
        assert ref.check_tolerance(y1, y_ref, bound, csr.val.dtype)[0]
        b0 = A.info()["build_seconds"]
        for k in (2, 3, 4, 7, 64):
            A.reencode(tpc=k)
            inf = A.info()
            assert inf["params"]["tiles_per_cta"] == k and inf["build_seconds"] == b0
            assert np.array_equal(_bits(A.spmv(x).cpu().numpy()), _bits(y1)), (k, name, p)
    finally:
        A.free()


def test_power_step_and_integer_exact():
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    csr = synth.webbase_like(m=200_000, integer=True)
    xn = synth.make_x(csr.n, np.float32, "int2", 5)
    x = torch.from_numpy(xn).cuda()
    y_ex = ref.spmv(csr.row_ptr, csr.col, csr.val, xn)[0]
    n2_in = torch.tensor([1.0], dtype=torch.float64, device="cuda")
    outs = []
    for k in (1, 2, 5):
        A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=0, T=8, C=64, tpc=k)
        y = A.spmv(x).cpu().numpy()
        assert np.array_equal(y.astype(np.float64), y_ex), k
        z = torch.empty(csr.m, dtype=torch.float32, device="cuda")
        n2 = torch.zeros(1, dtype=torch.float64, device="cuda")
        A.spmv_power(x, z, n2_in, n2)
        outs.append((z.cpu().numpy(), n2.item()))
        A.free()
    for z, n2 in outs[1:]:
        assert np.array_equal(z, outs[0][0]) and n2 == outs[0][1]


def test_auto_and_ticket_ids():
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    csr = synth.config_matrix("c4")
    A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=0, T=4, C=64)
    assert A.info()["params"]["tiles_per_cta"] in (1, 2)   # auto
    A.free()
    A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=0, T=4, C=64, tpc=4, flags=8)
    assert A.info()["params"]["tiles_per_cta"] == 1         # ticket ids: one tile per CTA
    A.free()
