"""__graft_entry__.smoke(): the driver's round-end check (one small fused
evaluation of c1 and c2/c3 samples on cuda:0 against the oracle)."""
import pytest

pytestmark = pytest.mark.gpu


def test_smoke():
    import __graft_entry__
    __graft_entry__.smoke()
