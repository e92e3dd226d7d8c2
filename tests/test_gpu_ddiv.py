"""The model kernel's branch-free division: wherever its range
test passes, the quotient is __ddiv_rn's bit pattern.  Random bit patterns
over the whole exponent range, model-like magnitudes, and the special and
boundary values around the two thresholds."""
import ctypes

import numpy as np
import pytest
import torch

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sel():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_chikinaat19_b200 as s
    return s


def _operands(seed):
    rng = np.random.default_rng(seed)
    n = 1 << 20
    bits = rng.integers(0, 2 ** 63, size=(2, n), dtype=np.uint64) | (rng.integers(0, 2, size=(2, n), dtype=np.uint64) << 63)
    a, b = bits.view(np.float64)
    # model-like magnitudes: cycles, bytes, clocks, weights in [1e-6, 1e15]
    m = n // 2
    a[:m] = 10.0 ** rng.uniform(-6, 15, m) * rng.choice([1, -1], m)
    b[:m] = 10.0 ** rng.uniform(-6, 15, m)
    # boundaries: a's high word near 2^-120, quotients near 2^-129 / 2^-1022, overflow, specials
    special = np.array([0.0, -0.0, np.inf, -np.inf, np.nan, 5e-324, 2.2250738585072014e-308, 1.0, -1.0, 3.0,
                        2.0 ** -120, 2.0 ** -121, 2.0 ** -119, 2.0 ** -129, 2.0 ** -1000, 2.0 ** 1000, 2.0 ** 1023,
                        1.7976931348623157e308, 2.0 ** -1022, 2.0 ** -1074, 7.0, 1e-300, 1e300])
    k = len(special)
    a[m:m + k * k] = np.repeat(special, k)
    b[m:m + k * k] = np.tile(special, k)
    j = m + k * k
    e = rng.integers(-1074, 1024, size=(2, 4096))
    a[j:j + 4096] = np.ldexp(rng.uniform(1, 2, 4096), e[0])
    b[j:j + 4096] = np.ldexp(rng.uniform(1, 2, 4096), e[1])
    return a, b


@pytest.mark.parametrize("seed", [1, 2])
def test_fast_division_matches_ddiv_rn(sel, seed):
    a, b = _operands(seed)
    n = len(a)
    da, db = torch.from_numpy(a).cuda(), torch.from_numpy(b).cuda()
    qf = torch.empty(n, dtype=torch.float64, device="cuda")
    qr = torch.empty_like(qf)
    ok = torch.empty(n, dtype=torch.uint8, device="cuda")
    L = sel._lib.lib()
    sel._lib.check(L.sel_selftest_ddiv(da.data_ptr(), db.data_ptr(), n, qf.data_ptr(), ok.data_ptr(),
                                       qr.data_ptr(), ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)))
    torch.cuda.synchronize()
    okh = ok.cpu().numpy().astype(bool)
    f = qf.cpu().numpy().view(np.uint64)
    r = qr.cpu().numpy().view(np.uint64)
    bad = np.nonzero(okh & (f != r))[0]
    assert len(bad) == 0, f"fast path differs at {bad[:5]}: a={a[bad[:5]]} b={b[bad[:5]]}"
    # the reference is IEEE division (numpy) wherever the fast path is taken
    with np.errstate(all="ignore"):
        ref = (a / b).view(np.uint64)
    assert (f[okh] == ref[okh]).all()
    # the fast path covers the model-like operands (it is the common case)
    assert okh[: n // 2].mean() > 0.999
