"""Host pin of the grid builder's coalescence links (CPU, no GPU): the number
of Eq.11 gathers per level (`lbm_grid_info.coal_links`) and of those with
|B| > 4 (`coal_wide`) counted by brute force from the masks, following
Stream(L) rule 5 as read in DESIGN.md §2 (R-A2, R-B1): a fluid leaf p at level
L and a direction e whose source s = p - e is REFINED form a gather when at
least one of the level-(L+1) cells 2p - e + {0,1}^3 is a fluid leaf.  The
velocity sets are written out here (independent of the library's tables)."""
import itertools

import numpy as np
import pytest

import lbm_inputs as I


def _velocities(Q):
    e = [c for c in itertools.product((-1, 0, 1), repeat=3) if any(c)]
    if Q == 19:
        e = [c for c in e if sum(abs(x) for x in c) <= 2]
    return np.array(e, dtype=np.int64)


def _brute_counts(prob):
    levels = prob.levels
    covered = [np.zeros(prob.level_shape(0), dtype=bool)]
    for L in range(1, levels):
        up = covered[L - 1] | (prob.masks[L - 1] != 0)
        covered.append(up.repeat(2, 0).repeat(2, 1).repeat(2, 2))
    links, wide = [], []
    for L in range(levels):
        if L + 1 >= levels:
            links.append(0)
            wide.append(0)
            continue
        m, mf = prob.masks[L], prob.masks[L + 1]
        refined = (m == 0) & ~covered[L]
        n = np.array(m.shape)
        nf = np.array(mf.shape)
        p = np.argwhere(m == 1)
        nl = nw = 0
        for e in _velocities(prob.Q):
            s = p - e
            ok = np.ones(len(p), dtype=bool)
            for a in range(3):
                if prob.periodic[a]:
                    s[:, a] %= n[a]
                else:
                    ok &= (s[:, a] >= 0) & (s[:, a] < n[a])
            sel = np.flatnonzero(ok)
            sel = sel[refined[s[sel, 0], s[sel, 1], s[sel, 2]]]
            cnt = np.zeros(len(sel), dtype=np.int64)
            for c in itertools.product((0, 1), repeat=3):
                b = 2 * p[sel] - e + np.array(c)
                okb = np.ones(len(sel), dtype=bool)
                for a in range(3):
                    if prob.periodic[a]:
                        b[:, a] %= nf[a]
                    else:
                        okb &= (b[:, a] >= 0) & (b[:, a] < nf[a])
                hit = np.zeros(len(sel), dtype=bool)
                idx = np.flatnonzero(okb)
                hit[idx] = mf[b[idx, 0], b[idx, 1], b[idx, 2]] == 1
                cnt += hit
            nl += int((cnt > 0).sum())
            nw += int((cnt > 4).sum())
        links.append(nl)
        wide.append(nw)
    return links, wide


PROBLEMS = {
    "cavity2": lambda: I.cavity2(),
    "random4": lambda: I.random_balanced(33, n=(9, 11, 10), levels=4, p_refine=0.5),
    "random_px": lambda: I.random_balanced(41, n=(12, 6, 6), levels=3, p_refine=0.6, periodic=(1, 0, 1)),
    "random_b": lambda: I.random_balanced(7, n=(10, 10, 10), levels=3, p_refine=0.5),
    "kbc_mini": lambda: I.cavity4_kbc("mini"),
    "tunnel_s5": lambda: I.tunnel4(scale=5),
}


@pytest.mark.parametrize("name", list(PROBLEMS))
def test_coalescence_link_counts_match_brute_force(name):
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    prob = PROBLEMS[name]()
    info = lbmr.analyze_problem(prob)
    links, wide = _brute_counts(prob)
    assert [int(info.coal_links[L]) for L in range(prob.levels)] == links
    assert [int(info.coal_wide[L]) for L in range(prob.levels)] == wide
    if name in ("random4", "random_px", "kbc_mini"):
        assert sum(wide) > 0  # the two-unit (|B| > 4) path is exercised by the GPU tests
