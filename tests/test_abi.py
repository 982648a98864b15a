"""The C-ABI library loads, exports every symbol include/yaspmv.h declares, and fails
loudly (no CPU fallback) on compute calls without a device.  CPU only."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    names = set()
    for h in sorted(os.listdir(os.path.join(ROOT, "include"))):
        src = open(os.path.join(ROOT, "include", h)).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        names |= set(re.findall(r"\b(yaspmv_[a-z0-9_]+)\s*\(", src))
    return sorted(names)


def test_every_declared_symbol_is_exported():
    import paper_conf_ppopp_yanlzz14_b200 as P
    from paper_conf_ppopp_yanlzz14_b200 import _lib
    names = _declared()
    assert len(names) >= 15
    assert sorted(names) == sorted(_lib.EXPORTED)
    out = subprocess.run(["nm", "-D", "--defined-only", _lib.LIB_PATH], capture_output=True, text=True).stdout
    for n in names:
        assert re.search(rf"\bT {n}$", out, re.M), n
        assert getattr(_lib.lib, n) is not None
    assert "sm_100a" in P.version()


def test_kernels_are_sm100a_cubins():
    from paper_conf_ppopp_yanlzz14_b200 import _lib
    out = subprocess.run(["cuobjdump", "--list-elf", _lib.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_host_only_handle_refuses_spmv():
    from paper_conf_ppopp_yanlzz14_b200 import Matrix, YaspmvError
    A = Matrix.from_csr(2, 2, np.array([0, 1, 2]), np.array([0, 1]), np.array([1.0, 2.0]), device=-1)
    with pytest.raises(YaspmvError) as e:
        A.spmv(0x1000, 0x2000, stream=0)
    assert e.value.status == 1 and "no CPU fallback" in str(e.value)


def test_argument_errors():
    from paper_conf_ppopp_yanlzz14_b200 import Matrix, YaspmvError
    rp = np.array([0, 1, 2]); c = np.array([0, 1]); v = np.array([1.0, 2.0])
    with pytest.raises(YaspmvError):
        Matrix.from_csr(2, 2, rp, np.array([0, 5]), v, device=-1)        # col out of range
    with pytest.raises(YaspmvError):
        Matrix.from_csr(2, 2, np.array([0, 2, 1]), c, v, device=-1)      # row_ptr not monotone
    with pytest.raises(YaspmvError):
        Matrix.from_csr(2, 2, rp, c, v, device=-1, h=5)                  # Table 1 range
    with pytest.raises(YaspmvError):
        Matrix.from_csr(2, 2, rp, c, v, device=-1, S=3)                  # S > NB
    with pytest.raises(YaspmvError):
        Matrix.from_csr(2, 70000, rp, c, v, device=-1, col_mode=1)       # u16 needs NB < 65535
    with pytest.raises(YaspmvError):
        Matrix.from_csr(2, 2, rp, c, v, device=-1, T=5)


def test_result_cache_parameter():
    """Table 1's strategy axis: result_cache 0 = strategy 1, {1,2,4} x C entries =
    strategy 2; other values are refused; the resolved value round-trips through get_info."""
    from paper_conf_ppopp_yanlzz14_b200 import Matrix, YaspmvError
    rp = np.array([0, 1, 2]); c = np.array([0, 1]); v = np.array([1.0, 2.0])
    for rc in (0, 1, 2, 4):
        A = Matrix.from_csr(2, 2, rp, c, v, device=-1, rc=rc)
        assert A.info()["params"]["result_cache"] == rc
        A.free()
    A = Matrix.from_csr(2, 2, rp, c, v, device=-1, rc=-1)
    assert A.info()["params"]["result_cache"] == 0
    A.free()
    for rc in (3, 5, 8):
        with pytest.raises(YaspmvError) as e:
            Matrix.from_csr(2, 2, rp, c, v, device=-1, rc=rc)
        assert e.value.status == 1


def test_tiles_per_cta_parameter():
    """tiles_per_cta: 0 = auto, 1..64 explicit, anything else refused (host-only handles
    report the requested value; device handles report the resolved one)."""
    from paper_conf_ppopp_yanlzz14_b200 import Matrix, YaspmvError
    rp = np.array([0, 1, 2]); c = np.array([0, 1]); v = np.array([1.0, 2.0])
    for k in (0, 1, 2, 64):
        A = Matrix.from_csr(2, 2, rp, c, v, device=-1, tpc=k)
        assert A.info()["params"]["tiles_per_cta"] == k
        A.free()
    for k in (-1, 65):
        with pytest.raises(YaspmvError) as e:
            Matrix.from_csr(2, 2, rp, c, v, device=-1, tpc=k)
        assert e.value.status == 1
