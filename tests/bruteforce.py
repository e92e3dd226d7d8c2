"""Independent pure-Python enumerator of the counting definition (a1-a3).

Used only to pin the C oracle on tiny inputs.  It is written from the
definition with a different loop structure from oracle.c: it walks the
parallel iterations p = 0..P-1 in order, derives (OpenMP repetition, block,
warp) of each iteration from the cyclic chunk-1 schedule (readings R6-R9),
groups iterations into warps with a dict, and counts distinct 128 B lines and
32 B sectors with Python sets over exact (big-int) addresses using Python's
floor division.  Nothing is shared with oracle.c.
"""
from __future__ import annotations

import itertools
from collections import OrderedDict

UNKNOWN = 0xFFFFFFFF


def counts(P0, P1, par_dims, trip, accesses, B, grid_max):
    """accesses: list of dicts {base, c_par (2), c_inner (3), elem, depth}.

    Returns (W, L, S, C, U, WR).
    """
    T = [128 if t == UNKNOWN else t for t in trip]
    P = P0 * P1
    if P == 0:
        return (0, 0, 0, 0, 0, 0)
    G = min(-(-P // B), grid_max)
    threads = G * B
    warps = OrderedDict()
    for p in range(P):
        rep, t = divmod(p, threads)
        blk, tid = divmod(t, B)
        warps.setdefault((rep, blk, tid // 32), []).append(p)
    W = L = S = C = U = 0
    for lanes in warps.values():
        for a in accesses:
            tmin = -(-32 * a["elem"] // 128)
            for idx in itertools.product(*[range(T[j]) for j in range(a["depth"])]):
                addrs = []
                for p in lanes:
                    if par_dims == 1:
                        x = a["base"] + a["c_par"][0] * p
                    else:
                        x = a["base"] + a["c_par"][0] * (p // P1) + a["c_par"][1] * (p % P1)
                    x += sum(a["c_inner"][j] * idx[j] for j in range(a["depth"]))
                    addrs.append(x)
                nl = len({x // 128 for x in addrs})
                ns = len({x // 32 for x in addrs})
                W += 1
                L += nl
                S += ns
                if nl <= tmin:
                    C += 1
                else:
                    U += nl
    return (W, L, S, C, U, len(warps))
