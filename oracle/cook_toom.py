"""ORACLE — TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Exact-rational Cook–Toom generator for the 1D Winograd minimal filter F(m, r),
written step by step from PAPER.md §5.3 (lines 586-603) and Figure 5
(lines 605-3179), in the paper's notation:

    Y = A^T [ (G g) ⊙ (D^T d) ]                     (Figure 1)

with alpha = m + r - 1 "states". The paper's D is
Lavin's B; we call D^T "BT". Shapes: AT is m x alpha, G is alpha x r,
BT is alpha x alpha. The result is a CORRELATION y_o = sum_k g_k d_{o+k}
(SURVEY.md §8(c) reading 1; pinned by tests against Figure 5).

Interpolation points: the alpha-1 finite points are taken in
order from 0, 1, -1, 2, -2, 1/2, -1/2, 3, -3, 1/3, -1/3, 4, -4, 1/4, -1/4
(the order of row 1 of A(16,15)^T); the last point is
infinity. DESIGN.md reading R7: for alpha = 16 the build also offers the
"alt" set 0, ±1, ±2, ±1/2, ±3, ±1/3, ±3/2, ±2/3 (same ± pairing, better fp32
conditioning); the paper's set stays here for the Figure-5 pin.

Steps:
  1. points a_0..a_{alpha-2} finite, a_{alpha-1} = infinity.
  2. AT[j][i] = a_i^j (j < m, i finite); AT[j][alpha-1] = [j == m-1].
  3. N_i = prod_{j != i} (a_i - a_j); G[i][k] = a_i^k / N_i; G[alpha-1][k] = [k == r-1].
  4. BT[i] = coefficients (degree 0..alpha-1) of M_i(x) = prod_{j != i}(x - a_j);
     BT[alpha-1] = coefficients of prod_j (x - a_j).
  5. Row-0 normalisation: move the factor 1/N_0 from G[0] to BT[0] so that
     G[0] = e_0 (a row scale moved between G and BT leaves the product unchanged).
"""
from __future__ import annotations

from fractions import Fraction as Fr

PAPER_POINTS = [Fr(0), Fr(1), Fr(-1), Fr(2), Fr(-2), Fr(1, 2), Fr(-1, 2), Fr(3), Fr(-3),
                Fr(1, 3), Fr(-1, 3), Fr(4), Fr(-4), Fr(1, 4), Fr(-1, 4)]
ALT16_POINTS = [Fr(0), Fr(1), Fr(-1), Fr(2), Fr(-2), Fr(1, 2), Fr(-1, 2), Fr(3), Fr(-3),
                Fr(1, 3), Fr(-1, 3), Fr(3, 2), Fr(-3, 2), Fr(2, 3), Fr(-2, 3)]


def finite_points(alpha: int, point_set: str = "paper"):
    src = PAPER_POINTS if point_set == "paper" else ALT16_POINTS
    if alpha - 1 > len(src):
        raise ValueError("alpha too large for the point list")
    return list(src[: alpha - 1])


def _poly_mul_linear(coeffs, a):
    """coeffs(x) * (x - a); coeffs low-degree first."""
    out = [Fr(0)] * (len(coeffs) + 1)
    for i, c in enumerate(coeffs):
        out[i + 1] += c
        out[i] -= a * c
    return out


def cook_toom(m: int, r: int, point_set: str = "paper"):
    """Return (AT, G, BT) as lists of lists of Fractions for F(m, r)."""
    alpha = m + r - 1
    pts = finite_points(alpha, point_set)
    nf = alpha - 1  # number of finite points
    # step 2: AT
    AT = [[Fr(0)] * alpha for _ in range(m)]
    for j in range(m):
        for i in range(nf):
            AT[j][i] = pts[i] ** j
        AT[j][alpha - 1] = Fr(1) if j == m - 1 else Fr(0)
    # step 3: G
    G = [[Fr(0)] * r for _ in range(alpha)]
    Ns = []
    for i in range(nf):
        Ni = Fr(1)
        for j in range(nf):
            if j != i:
                Ni *= pts[i] - pts[j]
        Ns.append(Ni)
        for k in range(r):
            G[i][k] = pts[i] ** k / Ni
    G[alpha - 1][r - 1] = Fr(1)
    # step 4: BT
    BT = []
    for i in range(nf):
        poly = [Fr(1)]
        for j in range(nf):
            if j != i:
                poly = _poly_mul_linear(poly, pts[j])
        poly = poly + [Fr(0)] * (alpha - len(poly))
        BT.append(poly)
    poly = [Fr(1)]
    for j in range(nf):
        poly = _poly_mul_linear(poly, pts[j])
    BT.append(poly + [Fr(0)] * (alpha - len(poly)))
    # step 5: row-0 normalisation (point 0 is always the first point)
    s = G[0][0]
    if s != 0:
        G[0] = [g / s for g in G[0]]
        BT[0] = [b * s for b in BT[0]]
    return AT, G, BT


def winograd_1d(AT, G, BT, g, d):
    """Y = AT [ (G g) ⊙ (BT d) ] in exact arithmetic (Figure 1)."""
    alpha = len(BT)
    u = [sum(G[i][k] * g[k] for k in range(len(g))) for i in range(alpha)]
    v = [sum(BT[i][j] * d[j] for j in range(alpha)) for i in range(alpha)]
    mm = [u[i] * v[i] for i in range(alpha)]
    return [sum(AT[o][i] * mm[i] for i in range(alpha)) for o in range(len(AT))]


def theoretical_acceleration(n: int, r: int) -> Fr:
    """Phi = n r / (n + r - 1)."""
    return Fr(n * r, n + r - 1)
