// Host-side 1-D reference tables for the CUDA path (independent of oracle/: different formulations).
//
//   Gauss-Legendre points/weights on [0,1], n = 2k (reading R3; PAPER.md:698-700 fixes 64 / 512 points
//       for 3D Q2 / Q4): Newton on P_n with the derivative recurrence P'_{j+1} = P'_{j-1} + (2j+1) P_j.
//   GLL nodes on [0,1], k+1 (reading R4): endpoints + Newton on f = P_{k-1} - x P_k  (= (1-x^2) P_k' / k).
//   Lagrange values/derivatives at the GL points: barycentric form.
//   Bernstein degree k-1 at the GL points (reading R5): de Casteljau-style recursion.
// Everything in long double, rounded once to double.
#pragma once
#include <cmath>
#include <vector>

namespace blastcf {

struct Tables1D {
  int k, n, p, t;
  std::vector<double> qpt, qwt, gll;   // [n], [n], [p]
  std::vector<double> B, G, Phi;       // [n][p], [n][p], [n][t]
};

inline void legendre_and_derivative(int n, long double x, long double &P, long double &dP) {
  // P_0 = 1, P_1 = x ; (j+1) P_{j+1} = (2j+1) x P_j - j P_{j-1} ; P'_{j+1} = P'_{j-1} + (2j+1) P_j
  long double pm = 1.0L, pc = x, dpm = 0.0L, dpc = 1.0L;
  if (n == 0) { P = 1.0L; dP = 0.0L; return; }
  for (int j = 1; j < n; ++j) {
    const long double pn = ((2.0L * j + 1.0L) * x * pc - (long double)j * pm) / (long double)(j + 1);
    const long double dpn = dpm + (2.0L * j + 1.0L) * pc;
    pm = pc; pc = pn; dpm = dpc; dpc = dpn;
  }
  P = pc; dP = dpc;
}

inline Tables1D build_tables(int k) {
  const long double pi = 3.141592653589793238462643383279502884L;
  Tables1D T;
  T.k = k; T.n = 2 * k; T.p = k + 1; T.t = k;
  const int n = T.n, p = T.p, t = T.t;
  std::vector<long double> xq(n), wq(n), xn(p);
  for (int i = 0; i < n; ++i) {
    long double x = -cosl(pi * (i + 0.75L) / (n + 0.5L));   // ascending initial guesses
    for (int it = 0; it < 60; ++it) {
      long double P, dP;
      legendre_and_derivative(n, x, P, dP);
      const long double dx = P / dP;
      x -= dx;
      if (fabsl(dx) <= 1e-28L) break;
    }
    long double P, dP;
    legendre_and_derivative(n, x, P, dP);
    xq[i] = 0.5L * (1.0L + x);
    wq[i] = 1.0L / ((1.0L - x * x) * dP * dP);   // 2/((1-x^2)P'^2) on [-1,1], halved on [0,1]
  }
  xn[0] = 0.0L;
  xn[k] = 1.0L;
  for (int i = 1; i < k; ++i) {
    long double x = -cosl(pi * i / k);
    for (int it = 0; it < 60; ++it) {
      long double Pk, dPk, Pk1, dPk1;
      legendre_and_derivative(k, x, Pk, dPk);
      legendre_and_derivative(k - 1, x, Pk1, dPk1);
      const long double f = Pk1 - x * Pk;
      const long double df = dPk1 - Pk - x * dPk;
      const long double dx = f / df;
      x -= dx;
      if (fabsl(dx) <= 1e-28L) break;
    }
    xn[i] = 0.5L * (1.0L + x);
  }
  // barycentric weights of the GLL nodes
  std::vector<long double> lam(p);
  for (int a = 0; a < p; ++a) {
    long double prod = 1.0L;
    for (int b = 0; b < p; ++b)
      if (b != a) prod *= (xn[a] - xn[b]);
    lam[a] = 1.0L / prod;
  }
  T.qpt.resize(n); T.qwt.resize(n); T.gll.resize(p);
  T.B.resize(n * p); T.G.resize(n * p); T.Phi.resize(n * t);
  for (int i = 0; i < n; ++i) { T.qpt[i] = (double)xq[i]; T.qwt[i] = (double)wq[i]; }
  for (int a = 0; a < p; ++a) T.gll[a] = (double)xn[a];
  for (int q = 0; q < n; ++q) {
    const long double xi = xq[q];
    long double den = 0.0L;
    for (int b = 0; b < p; ++b) den += lam[b] / (xi - xn[b]);
    for (int a = 0; a < p; ++a) {
      const long double la = (lam[a] / (xi - xn[a])) / den;
      long double s = 0.0L;
      for (int b = 0; b < p; ++b)
        if (b != a) s += 1.0L / (xi - xn[b]);
      T.B[q * p + a] = (double)la;
      T.G[q * p + a] = (double)(la * s);
    }
    // Bernstein of degree t-1 by the recursion b^m_j = (1-x) b^{m-1}_j + x b^{m-1}_{j-1}
    std::vector<long double> b(t, 0.0L);
    b[0] = 1.0L;
    for (int m = 1; m < t; ++m)
      for (int j = m; j >= 0; --j) b[j] = (1.0L - xi) * b[j] + (j > 0 ? xi * b[j - 1] : 0.0L);
    for (int j = 0; j < t; ++j) T.Phi[q * t + j] = (double)b[j];
  }
  return T;
}

// Monomial coefficients (in t = 2r - 1) of the degree-`deg` Chebyshev interpolant of
// y(r) = 2 cos(acos(r)/3), the largest root of y^3 - 3y - 2r = 0 on r in [0,1] (pointwise.cuh).
inline std::vector<double> eig_root_poly(int deg) {
  const long double pi = 3.141592653589793238462643383279502884L;
  const int n = deg + 1;
  std::vector<long double> f(n), c(n, 0.0L);
  for (int k = 0; k < n; ++k) {
    const long double t = cosl(pi * (k + 0.5L) / n), r = 0.5L * (t + 1.0L);
    f[k] = 2.0L * cosl(acosl(r) / 3.0L);
  }
  for (int j = 0; j < n; ++j) {
    long double s = 0.0L;
    for (int k = 0; k < n; ++k) s += f[k] * cosl(pi * j * (k + 0.5L) / n);
    c[j] = (j == 0 ? 1.0L : 2.0L) * s / n;
  }
  // sum_j c_j T_j(t) -> monomials, T_{j+1} = 2 t T_j - T_{j-1}
  std::vector<long double> mono(n, 0.0L), Tm(n, 0.0L), T0(n, 0.0L), T1(n, 0.0L);
  T0[0] = 1.0L;
  if (n > 1) T1[1] = 1.0L;
  for (int i = 0; i < n; ++i) mono[i] += c[0] * T0[i];
  if (n > 1)
    for (int i = 0; i < n; ++i) mono[i] += c[1] * T1[i];
  for (int j = 2; j < n; ++j) {
    for (int i = 0; i < n; ++i) Tm[i] = (i > 0 ? 2.0L * T1[i - 1] : 0.0L) - T0[i];
    for (int i = 0; i < n; ++i) mono[i] += c[j] * Tm[i];
    T0 = T1;
    T1 = Tm;
  }
  std::vector<double> out(n);
  for (int i = 0; i < n; ++i) out[i] = (double)mono[i];
  return out;
}

}  // namespace blastcf
