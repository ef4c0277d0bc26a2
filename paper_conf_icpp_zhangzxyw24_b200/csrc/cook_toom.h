// Host-side exact-rational Cook–Toom generator for 1D Winograd F(m, r)
// (row a0 of SURVEY.md §8(a)). Independent of oracle/ (shares no code).
//
// PAPER.md §5.3 (lines 586-603) and Figure 5 (605-3179):
//   Y = A^T [ (G g) ⊙ (D^T d) ],  alpha = m + r - 1 interpolation points,
//   alpha-1 finite points taken in order from
//   {0, 1, -1, 2, -2, 1/2, -1/2, 3, -3, 1/3, -1/3, 4, -4, 1/4, -1/4}, plus infinity.
//   A^T[j][i] = a_i^j, A^T[j][alpha-1] = [j == m-1]
//   N_i = prod_{j!=i}(a_i - a_j), G[i][k] = a_i^k / N_i, G[alpha-1][k] = [k == r-1]
//   D^T[i] = coeffs of prod_{j!=i}(x - a_j);  D^T[alpha-1] = coeffs of prod_j (x - a_j)
//   row 0 scaled so that G[0] = e_0 (the scale moves into D^T[0]).
// The product computes the CORRELATION y_o = sum_k g_k d_{o+k}.
// Point set 1 ("alt", alpha = 16 only, reading R7) replaces ±4, ±1/4 by
// ±3/2, ±2/3: same ± pairing, better fp32 conditioning.
#pragma once
#include <cstdint>
#include <cstdlib>
#include <stdexcept>
#include <vector>

namespace i2cw {

typedef __int128 i128;

inline i128 gcd128(i128 a, i128 b) {
  if (a < 0) a = -a;
  if (b < 0) b = -b;
  while (b) { i128 t = a % b; a = b; b = t; }
  return a;
}

struct Rat {
  i128 n = 0, d = 1;
  Rat() = default;
  Rat(long long v) : n(v), d(1) {}
  Rat(i128 a, i128 b) : n(a), d(b) { norm(); }
  void norm() {
    if (d == 0) throw std::runtime_error("cook_toom: zero denominator");
    if (d < 0) { n = -n; d = -d; }
    i128 g = gcd128(n, d);
    if (g > 1) { n /= g; d /= g; }
    const i128 lim = ((i128)1) << 100;  // overflow guard for the products below
    if (n > lim || n < -lim || d > lim) throw std::runtime_error("cook_toom: rational overflow");
  }
  double to_double() const { return (double)n / (double)d; }
};
inline Rat operator+(Rat a, Rat b) { i128 g = gcd128(a.d, b.d); return Rat(a.n * (b.d / g) + b.n * (a.d / g), a.d / g * b.d); }
inline Rat operator-(Rat a, Rat b) { return a + Rat(-b.n, b.d); }
inline Rat operator*(Rat a, Rat b) {
  i128 g1 = gcd128(a.n, b.d), g2 = gcd128(b.n, a.d);
  if (g1 == 0) g1 = 1;
  if (g2 == 0) g2 = 1;
  return Rat((a.n / g1) * (b.n / g2), (a.d / g2) * (b.d / g1));
}
inline Rat operator/(Rat a, Rat b) { return a * Rat(b.d, b.n); }
inline bool operator==(Rat a, Rat b) { return a.n == b.n && a.d == b.d; }

inline std::vector<Rat> finite_points(int alpha, int point_set) {
  static const long long paper[15][2] = {{0, 1}, {1, 1}, {-1, 1}, {2, 1}, {-2, 1}, {1, 2}, {-1, 2}, {3, 1},
                                         {-3, 1}, {1, 3}, {-1, 3}, {4, 1}, {-4, 1}, {1, 4}, {-1, 4}};
  static const long long alt[15][2] = {{0, 1}, {1, 1}, {-1, 1}, {2, 1}, {-2, 1}, {1, 2}, {-1, 2}, {3, 1},
                                       {-3, 1}, {1, 3}, {-1, 3}, {3, 2}, {-3, 2}, {2, 3}, {-2, 3}};
  if (alpha < 2 || alpha > 16) throw std::runtime_error("cook_toom: alpha out of range");
  std::vector<Rat> p;
  for (int i = 0; i < alpha - 1; ++i) {
    const long long* e = point_set == 1 ? alt[i] : paper[i];
    p.push_back(Rat((i128)e[0], (i128)e[1]));
  }
  return p;
}

struct Transforms {
  int m, r, alpha;
  std::vector<Rat> AT;  // m x alpha
  std::vector<Rat> G;   // alpha x r
  std::vector<Rat> BT;  // alpha x alpha
};

inline Rat rpow(Rat a, int e) { Rat v(1); for (int i = 0; i < e; ++i) v = v * a; return v; }

// coefficients (low degree first, length alpha) of prod_{j in idx} (x - a_j)
inline std::vector<Rat> poly_from_roots(const std::vector<Rat>& roots, int skip, int alpha) {
  std::vector<Rat> c(1, Rat(1));
  for (int j = 0; j < (int)roots.size(); ++j) {
    if (j == skip) continue;
    std::vector<Rat> o(c.size() + 1, Rat(0));
    for (size_t i = 0; i < c.size(); ++i) {
      o[i + 1] = o[i + 1] + c[i];
      o[i] = o[i] - roots[j] * c[i];
    }
    c.swap(o);
  }
  c.resize(alpha, Rat(0));
  return c;
}

inline Transforms cook_toom(int m, int r, int point_set) {
  if (m < 1 || r < 1) throw std::runtime_error("cook_toom: bad (m, r)");
  Transforms T;
  T.m = m; T.r = r; T.alpha = m + r - 1;
  const int a = T.alpha, nf = a - 1;
  std::vector<Rat> pts = finite_points(a, point_set);
  T.AT.assign((size_t)m * a, Rat(0));
  T.G.assign((size_t)a * r, Rat(0));
  T.BT.assign((size_t)a * a, Rat(0));
  for (int j = 0; j < m; ++j) {
    for (int i = 0; i < nf; ++i) T.AT[j * a + i] = rpow(pts[i], j);
    T.AT[j * a + a - 1] = Rat(j == m - 1 ? 1 : 0);
  }
  for (int i = 0; i < nf; ++i) {
    Rat Ni(1);
    for (int j = 0; j < nf; ++j)
      if (j != i) Ni = Ni * (pts[i] - pts[j]);
    for (int k = 0; k < r; ++k) T.G[i * r + k] = rpow(pts[i], k) / Ni;
    std::vector<Rat> c = poly_from_roots(pts, i, a);
    for (int k = 0; k < a; ++k) T.BT[i * a + k] = c[k];
  }
  T.G[(a - 1) * r + (r - 1)] = Rat(1);
  {
    std::vector<Rat> c = poly_from_roots(pts, -1, a);
    for (int k = 0; k < a; ++k) T.BT[(a - 1) * a + k] = c[k];
  }
  // row-0 normalisation: G[0] = e_0
  Rat s = T.G[0];
  if (!(s == Rat(0))) {
    for (int k = 0; k < r; ++k) T.G[k] = T.G[k] / s;
    for (int k = 0; k < a; ++k) T.BT[k] = T.BT[k] * s;
  }
  return T;
}

}  // namespace i2cw
