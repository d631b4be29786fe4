"""Host-only checks of the multi-GPU planning calls (bar_dist_ghosts / bar_dist_localize /
bar_dist_plan; no GPU): for random sparse matrices and random subdomain-aligned row partitions,
every rank's plan is consistent with every other rank's (what p sends to r is exactly what r
expects from p, in r's ghost order), ghost_src_idx points at the owner's row, and the local
numbering maps back to the global columns."""
import numpy as np
import pytest
from hypothesis import given, settings
from hypothesis import strategies as st

import workloads as W


def _D():
    from paper_conf_ipps_anzttdh12_b200 import dist as D

    return D


def _random_partition(rng, n, R, P):
    q = (n + R - 1) // R
    cuts = sorted(rng.choice(np.arange(1, q), size=min(P - 1, q - 1), replace=False).tolist()) if q > 1 else []
    bounds = [0] + [c * R for c in cuts] + [n]
    return [(bounds[i], bounds[i + 1]) for i in range(len(bounds) - 1)]


@settings(max_examples=25, deadline=None)
@given(seed=st.integers(0, 10_000), P=st.integers(1, 5), R=st.sampled_from([1, 7, 16, 64]))
def test_plans_are_mutually_consistent(seed, P, R):
    D = _D()
    rng = np.random.default_rng(seed)
    n = int(rng.integers(40, 400))
    A = W.random_dd(n, int(rng.integers(2, 8)), seed=seed, symmetric_pattern=bool(seed % 2))
    ranges = _random_partition(rng, n, R, P)
    P = len(ranges)
    blocks = []
    for a, c in ranges:
        s, e = A.rowptr[a], A.rowptr[c]
        blocks.append(W.CSR(n, (A.rowptr[a:c + 1] - s).astype(np.int32), A.col[s:e].copy(), A.val[s:e].copy(), a, c))
    gh = [D.ghosts(B) for B in blocks]
    glists = [np.concatenate(g) for g in gh]
    plans = [D.plan(r, ranges, glists) for r in range(P)]
    for r in range(P):
        rc, sc, si, gs = plans[r]
        b0, b1 = ranges[r]
        # ghosts: sorted, outside the owned rows, exactly the off-rank columns of the rows
        cols = blocks[r].col
        want = np.unique(cols[(cols < b0) | (cols >= b1)])
        assert np.array_equal(np.sort(glists[r]), want)
        assert rc.sum() == len(glists[r]) and rc[r] == 0 and sc[r] == 0
        # ghost_src: owner-local row of each ghost
        for j, c in enumerate(glists[r]):
            o = next(p for p, (a, e) in enumerate(ranges) if a <= c < e)
            assert gs[j] == c - ranges[o][0]
        # what r receives from p, in r's ghost order, is what p sends to r
        pos = 0
        for p in range(P):
            if p == r:
                continue
            got = glists[r][pos:pos + rc[p]]
            pos += rc[p]
            rc_p, sc_p, si_p, _ = plans[p]
            off = int(sc_p[:r].sum())
            sent = si_p[off:off + sc_p[r]] + ranges[p][0]
            assert np.array_equal(sent, got), (r, p)
        # local numbering maps back to the global columns, in order
        lo, hi = gh[r]
        cl = D.localize(blocks[r], lo, hi)
        back = np.where(cl < 0, np.concatenate([lo, [0]])[np.clip(cl + len(lo), 0, len(lo))],
                        np.where(cl >= b1 - b0, np.concatenate([hi, [0]])[np.clip(cl - (b1 - b0), 0, len(hi))],
                                 cl + b0))
        assert np.array_equal(back, cols)


def test_plan_errors():
    D = _D()
    with pytest.raises(D.BarError):  # a ghost column that no rank owns (ranges do not cover it)
        D.plan(0, [(0, 10), (10, 20)], [np.array([25], np.int32), np.zeros(0, np.int32)])
    with pytest.raises(D.BarError):  # non-contiguous row ranges
        D.plan(0, [(0, 10), (12, 20)], [np.zeros(0, np.int32), np.zeros(0, np.int32)])
