"""Pins of the oracle's NEXT rows against independent
numpy formulations.  CPU only."""
import numpy as np

import oracle


def test_select_launch_matches_numpy_argmin():
    rng = np.random.default_rng(3)
    n, G = 5000, 700
    group = rng.integers(0, G + 20, n).astype(np.uint32)          # some out-of-range groups
    t = rng.choice([0.5, 1.0, 2.0, np.inf], n) * rng.integers(1, 4, n)
    st = (rng.random(n) < 0.1).astype(np.uint8)
    best, val = oracle.select_launch(group, t, st, G)
    for g in range(G):
        idx = np.nonzero((group == g) & (st == 0))[0]
        if len(idx) == 0:
            assert best[g] == 0xFFFFFFFF and np.isinf(val[g])
            continue
        m = t[idx].min()
        first = idx[np.nonzero(t[idx] == m)[0][0]]                # ties: lowest index
        assert best[g] == first and val[g] == m
