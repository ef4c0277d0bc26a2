"""Pins for the oracle's exact Cook–Toom generator (oracle/cook_toom.py), -m "not gpu".

* entry-wise equality with the matrices printed in PAPER.md Figure 5 (tests/golden/fig5.txt);
* the exact identity A^T[(G g) ⊙ (B^T d)] == sum_k g_k d_{o+k} (1D correlation) with random
  rationals, for every (m, r) the build uses and both alpha=16 point sets;
* the worked F(2,3) example: d=[1,2,3,4], g=[1,1,1] -> y=[6,9];
* the pair structure of §5.3: rows (2k+1, 2k+2) agree at even positions
  and are opposite at odd positions;
* closed forms: Phi = nr/(n+r-1) and its maximum over r.
"""
import random
from fractions import Fraction as Fr

import pytest

from oracle.cook_toom import cook_toom, theoretical_acceleration, winograd_1d
from tests.golden_io import load_sections

PAIRS = [(7, 2), (6, 3), (5, 4), (4, 5), (3, 6), (2, 7),  # alpha 8
         (10, 7), (9, 8), (8, 9),                         # alpha 16
         (6, 7), (5, 8), (4, 9),                          # alpha 12
         (3, 2), (2, 3), (1, 4)]                          # alpha 4


def _parse(name):
    f = dict(kv.split("=") for kv in name.split()[1:] if "=" in kv)
    return name.split()[0], f


def test_figure5_entries():
    g = load_sections("fig5.txt")
    assert len(g) == 9
    for name, rows in g.items():
        kind, f = _parse(name)
        alpha = int(f["alpha"])
        sel = [int(t) for t in f["rows"].split(",")] if "rows" in f else range(len(rows))
        if kind == "AT":
            m = int(f["m"]); M = cook_toom(m, alpha - m + 1)[0]
        elif kind == "G":
            r = int(f["r"]); M = cook_toom(alpha - r + 1, r)[1]
        else:
            M = cook_toom(alpha - 1, 2)[2]
        for row, i in zip(rows, sel):
            assert M[i] == row, (name, i, M[i], row)


@pytest.mark.parametrize("m,r", PAIRS)
@pytest.mark.parametrize("pts", ["paper", "alt"])
def test_exact_correlation_identity(m, r, pts):
    if pts == "alt" and m + r - 1 != 16:
        pytest.skip("alt set only differs at alpha=16")
    AT, G, BT = cook_toom(m, r, pts)
    rnd = random.Random(m * 100 + r)
    for _ in range(3):
        g = [Fr(rnd.randint(-9, 9), rnd.randint(1, 5)) for _ in range(r)]
        d = [Fr(rnd.randint(-9, 9), rnd.randint(1, 5)) for _ in range(m + r - 1)]
        y = winograd_1d(AT, G, BT, g, d)
        assert y == [sum(g[k] * d[o + k] for k in range(r)) for o in range(m)]


def test_worked_f23():
    AT, G, BT = cook_toom(2, 3)
    d = [Fr(1), Fr(2), Fr(3), Fr(4)]
    assert [sum(BT[i][j] * d[j] for j in range(4)) for i in range(4)] == [-2, 5, 1, 2]
    assert [sum(G[i][k] for k in range(3)) for i in range(4)] == [1, Fr(3, 2), Fr(1, 2), 1]
    assert winograd_1d(AT, G, BT, [1, 1, 1], d) == [6, 9]
    assert winograd_1d(AT, G, BT, [1, 2, 3], d) == [14, 20]


@pytest.mark.parametrize("m,r", PAIRS)
def test_pair_symmetry(m, r):
    AT, G, BT = cook_toom(m, r, "alt" if m + r - 1 == 16 else "paper")
    alpha = m + r - 1
    for k in range((alpha - 2) // 2):
        a, b = 2 * k + 1, 2 * k + 2
        for j in range(alpha):
            s = 1 if j % 2 == 0 else -1
            assert BT[b][j] == s * BT[a][j]
        for j in range(r):
            s = 1 if j % 2 == 0 else -1
            assert G[b][j] == s * G[a][j]
        for o in range(m):
            s = 1 if o % 2 == 0 else -1
            assert AT[o][b] == s * AT[o][a]


def test_theoretical_acceleration():
    assert theoretical_acceleration(6, 3) == Fr(18, 8)
    for alpha in (4, 8, 16):
        best = max(theoretical_acceleration(alpha - r + 1, r) for r in range(2, alpha))
        # even alpha reaches ceil((a+1)/2) floor((a+1)/2) / alpha
        assert best == Fr(((alpha + 2) // 2) * ((alpha + 1) // 2), alpha)
