/*
 * oracle/blast_oracle.c — CPU ORACLE for the BLAST corner force.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load this library.  The product path (paper_conf_ipps_dongdkrtd14_b200/) never links, imports
 * or calls it, and it shares no code, header, table or constant generator with csrc/.
 *
 * What it computes (§2, eqs (4)-(6)): for every zone z the generalized corner
 * force matrix
 *     (F_z)_{(c,a), j} = sum_q alpha_q  sum_d S_cd(q) dW_a/dxi_d(q)  phi_j(q),
 *     S(q) = sigma(q) adj(J_z(q))^T          ( = alpha-less  sigma : J^{-1} grad W |J| ),
 * i.e. F_z = A_z B^T with (A_z)_{(c,a),q} = alpha_q sum_d S_cd dW_a/dxi_d (eq 5) and
 * B_{jq} = phi_j(q) (eq 6), and from it the two right-hand sides the integrator needs
 * (eqs (1)-(2); kernels 8 and 10):
 *     F.1   assembled into global kinematic DOFs, serially in ascending zone id,
 *     F_z^T V_z per zone,
 * and the minimum time-step estimate over zones and quadrature points (steps 4.2 and 5 of the
 * BLAST algorithm).
 *
 * The stress sigma(q) "involves SVD, eigenvalue, eigenvector, EOS" and is
 * defined in ref. [1]; the constants and formulas used here are the readings listed in
 * DESIGN.md §3 (ideal-gas EOS, tensor artificial viscosity with compression length scale and
 * vorticity switch, dt from the smallest singular value of J).  Parity of the viscous terms is
 * pinned by closed forms (dt at rest, uniform expansion) and by invariants; the general viscous
 * stress is "parity unpinned" against the paper itself (its constants are a reading).
 *
 * Plain and slow on purpose: dense reference-element tables, every quadrature point evaluated
 * from the definition, eigenpairs by cyclic Jacobi, no sum factorization, no fusion.  Compiled
 * with -O2 -fno-fast-math -ffp-contract=off.  OpenMP parallelism is over zones only; assembly is
 * serial.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

typedef long double ld;

/* ------------------------------------------------------------------------------------------ */
/* 1-D tables on the reference segment [0,1] (reading DESIGN.md R3, R4, R5, R14)             */
/* ------------------------------------------------------------------------------------------ */

/* Legendre P_n and P_n' at x in [-1,1] by the three-term recurrence. */
static void legendre(int n, ld x, ld *P, ld *dP) {
  ld p0 = 1.0L, p1 = x;
  if (n == 0) { *P = 1.0L; *dP = 0.0L; return; }
  for (int j = 1; j < n; ++j) {
    ld p2 = ((2.0L * j + 1.0L) * x * p1 - (ld)j * p0) / (ld)(j + 1);
    p0 = p1;
    p1 = p2;
  }
  *P = p1;
  /* P_n'(x) = n (x P_n - P_{n-1}) / (x^2 - 1), valid for |x| < 1 */
  *dP = (ld)n * (x * p1 - p0) / (x * x - 1.0L);
}

/* Gauss-Legendre points/weights on [0,1]: Newton on P_n (long double). */
void oracle_gauss_legendre01(int n, double *pts, double *wts) {
  for (int i = 0; i < n; ++i) {
    ld x = cosl(3.14159265358979323846264338327950288L * ((ld)i + 0.75L) / ((ld)n + 0.5L));
    for (int it = 0; it < 100; ++it) {
      ld P, dP;
      legendre(n, x, &P, &dP);
      ld dx = P / dP;
      x -= dx;
      if (fabsl(dx) < 1e-30L) break;
    }
    ld P, dP;
    legendre(n, x, &P, &dP);
    ld w = 2.0L / ((1.0L - x * x) * dP * dP);
    /* x_i descending in [-1,1]; store ascending on [0,1] */
    pts[n - 1 - i] = (double)(0.5L * (x + 1.0L));
    wts[n - 1 - i] = (double)(0.5L * w);
  }
}

/* Same, kept in long double for the oracle's own tables. */
static void gauss_legendre01_ld(int n, ld *pts, ld *wts) {
  for (int i = 0; i < n; ++i) {
    ld x = cosl(3.14159265358979323846264338327950288L * ((ld)i + 0.75L) / ((ld)n + 0.5L));
    for (int it = 0; it < 100; ++it) {
      ld P, dP;
      legendre(n, x, &P, &dP);
      ld dx = P / dP;
      x -= dx;
      if (fabsl(dx) < 1e-30L) break;
    }
    ld P, dP;
    legendre(n, x, &P, &dP);
    pts[n - 1 - i] = 0.5L * (x + 1.0L);
    wts[n - 1 - i] = 0.5L * 2.0L / ((1.0L - x * x) * dP * dP);
  }
}

/* Gauss-Lobatto-Legendre nodes on [0,1], k+1 of them: 0, roots of P_k', 1 (Newton, long double). */
static void gll01_ld(int k, ld *nodes) {
  nodes[0] = 0.0L;
  nodes[k] = 1.0L;
  for (int i = 1; i < k; ++i) {
    ld x = -cosl(3.14159265358979323846264338327950288L * (ld)i / (ld)k);
    for (int it = 0; it < 100; ++it) {
      ld P, dP;
      legendre(k, x, &P, &dP);
      /* Legendre ODE: (1-x^2) P'' = 2x P' - k(k+1) P */
      ld d2P = (2.0L * x * dP - (ld)k * (ld)(k + 1) * P) / (1.0L - x * x);
      ld dx = dP / d2P;
      x -= dx;
      if (fabsl(dx) < 1e-30L) break;
    }
    nodes[i] = 0.5L * (x + 1.0L);
  }
}

void oracle_gll01(int k, double *nodes) {
  ld t[16];
  gll01_ld(k, t);
  for (int i = 0; i <= k; ++i) nodes[i] = (double)t[i];
}

/* Lagrange basis on nodes[0..np-1] at xi: values and derivatives (plain product formulas). */
static void lagrange_ld(int np, const ld *nodes, ld xi, ld *val, ld *der) {
  for (int a = 0; a < np; ++a) {
    ld v = 1.0L;
    for (int b = 0; b < np; ++b)
      if (b != a) v *= (xi - nodes[b]) / (nodes[a] - nodes[b]);
    val[a] = v;
    ld d = 0.0L;
    for (int m = 0; m < np; ++m) {
      if (m == a) continue;
      ld term = 1.0L / (nodes[a] - nodes[m]);
      for (int b = 0; b < np; ++b)
        if (b != a && b != m) term *= (xi - nodes[b]) / (nodes[a] - nodes[b]);
      d += term;
    }
    der[a] = d;
  }
}

/* Bernstein polynomials of degree m on [0,1] at xi: C(m,j) xi^j (1-xi)^(m-j). */
static void bernstein_ld(int m, ld xi, ld *val) {
  for (int j = 0; j <= m; ++j) {
    ld c = 1.0L;
    for (int i = 0; i < j; ++i) c = c * (ld)(m - i) / (ld)(i + 1);
    val[j] = c * powl(xi, (ld)j) * powl(1.0L - xi, (ld)(m - j));
  }
}

/* Export the 1-D tables for the table pins (tests/test_oracle_tables.py).
 * qpt,qwt [n=2k]; gll [k+1]; B,G [n][k+1] (W_a, W_a' at qp); Phi [n][k] (Bernstein deg k-1). */
void oracle_tables_1d(int k, double *qpt, double *qwt, double *gll, double *B, double *G, double *Phi) {
  int n = 2 * k, p = k + 1;
  ld xq[32], wq[32], xn[16], val[16], der[16];
  gauss_legendre01_ld(n, xq, wq);
  gll01_ld(k, xn);
  for (int i = 0; i < n; ++i) { qpt[i] = (double)xq[i]; qwt[i] = (double)wq[i]; }
  for (int a = 0; a < p; ++a) gll[a] = (double)xn[a];
  for (int q = 0; q < n; ++q) {
    lagrange_ld(p, xn, xq[q], val, der);
    for (int a = 0; a < p; ++a) { B[q * p + a] = (double)val[a]; G[q * p + a] = (double)der[a]; }
    bernstein_ld(k - 1, xq[q], val);
    for (int j = 0; j < k; ++j) Phi[q * k + j] = (double)val[j];
  }
}

/* ------------------------------------------------------------------------------------------ */
/* Dense reference-element tables: W_a(q), dW_a/dxi_d(q), phi_j(q), alpha_q                    */
/* ------------------------------------------------------------------------------------------ */
typedef struct {
  int dim, k, n, p, nq, nk, nt;
  double *alpha; /* [nq] */
  double *dW;    /* [nq][nk][dim] */
  double *phi;   /* [nq][nt] */
} tables_t;

static int ipow(int b, int e) { int r = 1; while (e-- > 0) r *= b; return r; }

static int tables_build(tables_t *T, int dim, int k) {
  T->dim = dim; T->k = k; T->n = 2 * k; T->p = k + 1;
  T->nq = ipow(T->n, dim); T->nk = ipow(T->p, dim); T->nt = ipow(k, dim);
  T->alpha = (double *)malloc(sizeof(double) * T->nq);
  T->dW = (double *)malloc(sizeof(double) * (size_t)T->nq * T->nk * dim);
  T->phi = (double *)malloc(sizeof(double) * (size_t)T->nq * T->nt);
  if (!T->alpha || !T->dW || !T->phi) return -1;
  int n = T->n, p = T->p;
  ld xq[32], wq[32], xn[16];
  ld B[32][16], G[32][16], Ph[32][16];
  gauss_legendre01_ld(n, xq, wq);
  gll01_ld(k, xn);
  for (int q = 0; q < n; ++q) {
    lagrange_ld(p, xn, xq[q], B[q], G[q]);
    bernstein_ld(k - 1, xq[q], Ph[q]);
  }
  for (int q = 0; q < T->nq; ++q) {
    int qi[3] = {q % n, (q / n) % n, (q / (n * n)) % n};
    ld w = 1.0L;
    for (int t = 0; t < dim; ++t) w *= wq[qi[t]];
    T->alpha[q] = (double)w;
    for (int a = 0; a < T->nk; ++a) {
      int ai[3] = {a % p, (a / p) % p, (a / (p * p)) % p};
      for (int d = 0; d < dim; ++d) {
        ld g = 1.0L;
        for (int t = 0; t < dim; ++t) g *= (t == d) ? G[qi[t]][ai[t]] : B[qi[t]][ai[t]];
        T->dW[((size_t)q * T->nk + a) * dim + d] = (double)g;
      }
    }
    for (int j = 0; j < T->nt; ++j) {
      int ji[3] = {j % k, (j / k) % k, (j / (k * k)) % k};
      ld f = 1.0L;
      for (int t = 0; t < dim; ++t) f *= Ph[qi[t]][ji[t]];
      T->phi[(size_t)q * T->nt + j] = (double)f;
    }
  }
  return 0;
}

static void tables_free(tables_t *T) { free(T->alpha); free(T->dW); free(T->phi); }

/* ------------------------------------------------------------------------------------------ */
/* Small dense linear algebra, d = 2 or 3                                                      */
/* ------------------------------------------------------------------------------------------ */
static double det_d(int d, const double M[3][3]) {
  if (d == 2) return M[0][0] * M[1][1] - M[0][1] * M[1][0];
  return M[0][0] * (M[1][1] * M[2][2] - M[1][2] * M[2][1]) - M[0][1] * (M[1][0] * M[2][2] - M[1][2] * M[2][0]) +
         M[0][2] * (M[1][0] * M[2][1] - M[1][1] * M[2][0]);
}

/* adjugate (transpose of the cofactor matrix): M adj(M) = det(M) I */
static void adj_d(int d, const double M[3][3], double A[3][3]) {
  if (d == 2) {
    A[0][0] = M[1][1]; A[0][1] = -M[0][1];
    A[1][0] = -M[1][0]; A[1][1] = M[0][0];
    return;
  }
  A[0][0] = M[1][1] * M[2][2] - M[1][2] * M[2][1];
  A[0][1] = M[0][2] * M[2][1] - M[0][1] * M[2][2];
  A[0][2] = M[0][1] * M[1][2] - M[0][2] * M[1][1];
  A[1][0] = M[1][2] * M[2][0] - M[1][0] * M[2][2];
  A[1][1] = M[0][0] * M[2][2] - M[0][2] * M[2][0];
  A[1][2] = M[0][2] * M[1][0] - M[0][0] * M[1][2];
  A[2][0] = M[1][0] * M[2][1] - M[1][1] * M[2][0];
  A[2][1] = M[0][1] * M[2][0] - M[0][0] * M[2][1];
  A[2][2] = M[0][0] * M[1][1] - M[0][1] * M[1][0];
}

/* Symmetric eigen-decomposition by cyclic Jacobi rotations (Golub & Van Loan §8.5).
 * Eigenvalues ascending in lam[]; column i of V (V[.][i]) is the unit eigenvector of lam[i].
 * Exact ties keep the lower coordinate index first (stable sort), so a scalar matrix gives
 * V = I and the "smallest" eigenvector e_1 (reading DESIGN.md R9). */
void oracle_sym_eig(int d, const double *Ain, double *lam, double *Vout) {
  double A[3][3], V[3][3];
  for (int i = 0; i < d; ++i)
    for (int j = 0; j < d; ++j) { A[i][j] = Ain[i * d + j]; V[i][j] = (i == j) ? 1.0 : 0.0; }
  for (int sweep = 0; sweep < 100; ++sweep) {
    double off = 0.0;
    for (int i = 0; i < d; ++i)
      for (int j = i + 1; j < d; ++j) off += A[i][j] * A[i][j];
    if (off == 0.0) break;
    for (int pp = 0; pp < d; ++pp) {
      for (int qq = pp + 1; qq < d; ++qq) {
        double apq = A[pp][qq];
        if (apq == 0.0) continue;
        /* negligible off-diagonal entry: drop it (classical threshold) */
        if (fabs(apq) <= 1e-300 || (fabs(A[pp][pp]) + fabs(apq) * 1e18 == fabs(A[pp][pp]) &&
                                    fabs(A[qq][qq]) + fabs(apq) * 1e18 == fabs(A[qq][qq]))) {
          A[pp][qq] = A[qq][pp] = 0.0;
          continue;
        }
        double theta = (A[qq][qq] - A[pp][pp]) / (2.0 * apq);
        double t;
        if (fabs(theta) > 1e150) t = 0.5 / theta;
        else t = (theta >= 0.0 ? 1.0 : -1.0) / (fabs(theta) + sqrt(theta * theta + 1.0));
        double c = 1.0 / sqrt(t * t + 1.0), s = t * c;
        /* A <- R^T A R with R the rotation in the (pp,qq) plane */
        for (int r = 0; r < d; ++r) {
          double arp = A[r][pp], arq = A[r][qq];
          A[r][pp] = c * arp - s * arq;
          A[r][qq] = s * arp + c * arq;
        }
        for (int r = 0; r < d; ++r) {
          double apr = A[pp][r], aqr = A[qq][r];
          A[pp][r] = c * apr - s * aqr;
          A[qq][r] = s * apr + c * aqr;
        }
        A[pp][qq] = A[qq][pp] = 0.0;
        for (int r = 0; r < d; ++r) {
          double vrp = V[r][pp], vrq = V[r][qq];
          V[r][pp] = c * vrp - s * vrq;
          V[r][qq] = s * vrp + c * vrq;
        }
      }
    }
  }
  int idx[3] = {0, 1, 2};
  double ev[3];
  for (int i = 0; i < d; ++i) ev[i] = A[i][i];
  /* stable insertion sort ascending */
  for (int i = 1; i < d; ++i) {
    int j = i;
    while (j > 0 && ev[idx[j - 1]] > ev[idx[j]]) { int tmp = idx[j]; idx[j] = idx[j - 1]; idx[j - 1] = tmp; --j; }
  }
  for (int i = 0; i < d; ++i) {
    lam[i] = ev[idx[i]];
    for (int r = 0; r < d; ++r) Vout[r * d + i] = V[r][idx[i]];
  }
}

/* Smallest singular value of J: sqrt of the smallest eigenvalue of J^T J. */
double oracle_sigma_min(int d, const double *J) {
  double JtJ[9], lam[3], V[9];
  for (int i = 0; i < d; ++i)
    for (int j = 0; j < d; ++j) {
      double s = 0.0;
      for (int r = 0; r < d; ++r) s += J[r * d + i] * J[r * d + j];
      JtJ[i * d + j] = s;
    }
  oracle_sym_eig(d, JtJ, lam, V);
  return sqrt(lam[0] > 0.0 ? lam[0] : 0.0);
}

/* smooth step of the viscosity compression switch (reading DESIGN.md R8) */
static double smooth_step01(double x, double eps) {
  double y = (x + eps) / (2.0 * eps);
  if (y < 0.0) return 0.0;
  if (y > 1.0) return 1.0;
  return (3.0 - 2.0 * y) * y * y;
}

/* ------------------------------------------------------------------------------------------ */
/* The corner force                                                                            */
/* ------------------------------------------------------------------------------------------ */

/* params[] = { cfl, q_quad, q_lin, eps_switch, h0, use_viscosity, use_vorticity } */
enum { P_CFL = 0, P_QQUAD, P_QLIN, P_EPS, P_H0, P_VISC, P_VORT, P_COUNT };

/* Total initial volume sum_z sum_q alpha_q det J0(z,q) (used by h0, reading R11). */
double oracle_volume(int dim, int k, int64_t Z, const int32_t *zone_nodes, int64_t nnodes, const double *x0) {
  tables_t T;
  if (tables_build(&T, dim, k)) return -1.0;
  double vol = 0.0;
  for (int64_t z = 0; z < Z; ++z) {
    for (int q = 0; q < T.nq; ++q) {
      double J[3][3] = {{0}};
      for (int a = 0; a < T.nk; ++a) {
        int64_t node = zone_nodes[z * T.nk + a];
        for (int c = 0; c < dim; ++c)
          for (int d = 0; d < dim; ++d) J[c][d] += x0[c * nnodes + node] * T.dW[((size_t)q * T.nk + a) * dim + d];
      }
      vol += T.alpha[q] * det_d(dim, J);
    }
  }
  tables_free(&T);
  return vol;
}

/* diag[] per run: 0 min det J, 1 min relative eigen-gap of eps ((l1-l0)/||eps||_F where eps != 0),
 *                 2 min |lambda - 2 eps_sw|, 3 #qps with inv_dt <= 0, 4 #qps with det J <= 0 */
enum { D_MINDET = 0, D_MINGAP, D_MINSW, D_NOINV, D_NBAD, D_COUNT };

/*
 * Evaluate the corner force on zones zone_list[0..nsub-1] (ascending; NULL = all Z zones).
 *   x, v, x0     [dim][nnodes]      e [Z][nt]      rho0detJ0 [Z][nq] (no quadrature weight)
 *   zone_gamma   [Z]
 * Outputs (any may be NULL):
 *   out_F1       [dim][nnodes]  assembled F.1 over the evaluated zones (serial, ascending zone)
 *   out_Fz1      [nsub][dim][nk] zone-local F_z.1
 *   out_FTv      [nsub][nt]     F_z^T V_z
 *   out_dtz      [nsub]         per-zone dt (0 if some det J <= 0, +inf if no qp has inv_dt > 0)
 *   out_dt_min   [1]            min of out_dtz
 *   out_Fz       [nsub][dim*nk][nt]  if non-NULL: "definition mode" — F_z = A_z B^T is formed and
 *                F.1, F^T v are taken from it (kernels 7, 8, 10).  Otherwise
 *                F_z.1 = A_z (B^T 1) and F_z^T V = B (A_z^T V) (associativity of eq (5)-(6)).
 *   diag         [D_COUNT]
 * Returns 0, or -1 on allocation failure / bad arguments.
 */
int oracle_eval(int dim, int k, int64_t Z, int64_t nnodes, const int32_t *zone_nodes, const double *x,
                const double *v, const double *e, const double *rho0detJ0, const double *x0,
                const double *zone_gamma, const double *params, const int64_t *zone_list, int64_t nsub,
                double *out_F1, double *out_Fz1, double *out_FTv, double *out_dtz, double *out_dt_min,
                double *out_Fz, double *diag, int nthreads) {
  if (dim < 2 || dim > 3 || k < 1 || k > 8) return -1;
  tables_t T;
  if (tables_build(&T, dim, k)) return -1;
  const int nq = T.nq, nk = T.nk, nt = T.nt, dk = dim * nk;
  if (!zone_list) nsub = Z;
  const double cfl = params[P_CFL], q_quad = params[P_QQUAD], q_lin = params[P_QLIN], eps_sw = params[P_EPS];
  const int use_visc = params[P_VISC] != 0.0, use_vort = params[P_VORT] != 0.0;
  double h0 = params[P_H0];
  if (!(h0 > 0.0)) {
    double vol = oracle_volume(dim, k, Z, zone_nodes, nnodes, x0);
    h0 = pow(vol / (double)Z, 1.0 / dim) / (double)k;
  }
  double *Fz1_all = (double *)malloc(sizeof(double) * (size_t)nsub * dk);
  double *dt_all = (double *)malloc(sizeof(double) * (size_t)nsub);
  double *dg_all = (double *)malloc(sizeof(double) * (size_t)nsub * D_COUNT);
  if (!Fz1_all || !dt_all || !dg_all) { tables_free(&T); free(Fz1_all); free(dt_all); free(dg_all); return -1; }
  int failed = 0;
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#pragma omp parallel
#endif
  {
    double *X = (double *)malloc(sizeof(double) * dk);
    double *Vz = (double *)malloc(sizeof(double) * dk);
    double *X0 = (double *)malloc(sizeof(double) * dk);
    double *Acol = (double *)malloc(sizeof(double) * dk);
    double *FTv = (double *)malloc(sizeof(double) * nt);
    double *Fz = out_Fz ? (double *)malloc(sizeof(double) * (size_t)dk * nt) : NULL;
    if (!X || !Vz || !X0 || !Acol || !FTv || (out_Fz && !Fz)) {
#ifdef _OPENMP
#pragma omp atomic write
#endif
      failed = 1;
    } else {
#ifdef _OPENMP
#pragma omp for schedule(dynamic, 4)
#endif
      for (int64_t s = 0; s < nsub; ++s) {
        const int64_t z = zone_list ? zone_list[s] : s;
        double *Fz1 = Fz1_all + (size_t)s * dk;
        double *dg = dg_all + (size_t)s * D_COUNT;
        dg[D_MINDET] = INFINITY; dg[D_MINGAP] = INFINITY; dg[D_MINSW] = INFINITY;
        dg[D_NOINV] = 0.0; dg[D_NBAD] = 0.0;
        /* gather X_z, V_z, X0_z through the zone -> node map */
        for (int a = 0; a < nk; ++a) {
          int64_t node = zone_nodes[z * nk + a];
          for (int c = 0; c < dim; ++c) {
            X[c * nk + a] = x[c * nnodes + node];
            Vz[c * nk + a] = v[c * nnodes + node];
            X0[c * nk + a] = x0[c * nnodes + node];
          }
        }
        const double *Ez = e + z * nt;
        const double gamma = zone_gamma[z];
        for (int i = 0; i < dk; ++i) Fz1[i] = 0.0;
        for (int j = 0; j < nt; ++j) FTv[j] = 0.0;
        if (Fz) for (int i = 0; i < dk * nt; ++i) Fz[i] = 0.0;
        double dtz = INFINITY;
        int bad = 0;
        for (int q = 0; q < nq; ++q) {
          const double *dWq = T.dW + (size_t)q * nk * dim;
          const double *phq = T.phi + (size_t)q * nt;
          /* step 1: J = X_z grad W (J_cd = dx_c/dxi_d), det, adjugate, inverse */
          double J[3][3] = {{0}}, J0[3][3] = {{0}}, gvh[3][3] = {{0}};
          for (int a = 0; a < nk; ++a)
            for (int c = 0; c < dim; ++c)
              for (int d = 0; d < dim; ++d) J[c][d] += X[c * nk + a] * dWq[a * dim + d];
          const double detJ = det_d(dim, J);
          double adjJ[3][3], Jinv[3][3];
          adj_d(dim, J, adjJ);
          for (int c = 0; c < dim; ++c)
            for (int d = 0; d < dim; ++d) Jinv[c][d] = adjJ[c][d] / detJ;
          if (detJ < dg[D_MINDET]) dg[D_MINDET] = detJ;
          if (detJ <= 0.0) { bad = 1; dg[D_NBAD] += 1.0; }
          /* step 3: EOS at the qp: rho = rho0|J0| / |J|, e(q) = sum_j E_j phi_j(q) clamped >= 0 */
          const double rho = rho0detJ0[z * nq + q] / detJ;
          double eq = 0.0;
          for (int j = 0; j < nt; ++j) eq += Ez[j] * phq[j];
          if (eq < 0.0) eq = 0.0;
          const double pres = (gamma - 1.0) * rho * eq;
          const double cs = sqrt(gamma * (gamma - 1.0) * eq);
          double sigma[3][3] = {{0}};
          for (int c = 0; c < dim; ++c) sigma[c][c] = -pres;
          double mu = 0.0;
          /* step 2: velocity gradient and artificial viscosity */
          if (use_visc) {
            for (int a = 0; a < nk; ++a)
              for (int c = 0; c < dim; ++c)
                for (int d = 0; d < dim; ++d) gvh[c][d] += Vz[c * nk + a] * dWq[a * dim + d];
            double gv[3][3];
            for (int c = 0; c < dim; ++c)
              for (int f = 0; f < dim; ++f) {
                double s = 0.0;
                for (int d = 0; d < dim; ++d) s += gvh[c][d] * Jinv[d][f];
                gv[c][f] = s;
              }
            double psi0 = 1.0;
            if (use_vort) {
              double tr = 0.0, fn = 0.0;
              for (int c = 0; c < dim; ++c) tr += gv[c][c];
              for (int c = 0; c < dim; ++c)
                for (int f = 0; f < dim; ++f) fn += gv[c][f] * gv[c][f];
              fn = sqrt(fn);
              psi0 = (fn > 0.0) ? fabs(tr) / fn : 1.0;
            }
            double eps[9], lam[3], vec[9];
            double fe = 0.0;
            for (int c = 0; c < dim; ++c)
              for (int f = 0; f < dim; ++f) {
                eps[c * dim + f] = 0.5 * (gv[c][f] + gv[f][c]);
                fe += eps[c * dim + f] * eps[c * dim + f];
              }
            oracle_sym_eig(dim, eps, lam, vec);
            fe = sqrt(fe);
            if (fe > 0.0) {
              double gap = (lam[1] - lam[0]) / fe;
              if (gap < dg[D_MINGAP]) dg[D_MINGAP] = gap;
            }
            double dsw = fabs(lam[0] - 2.0 * eps_sw);
            if (dsw < dg[D_MINSW]) dg[D_MINSW] = dsw;
            /* compression direction s = eigenvector of the smallest eigenvalue; length scale
               l = h0 |J J0^{-1} s| with J0 the initial Jacobian at the same point */
            for (int a = 0; a < nk; ++a)
              for (int c = 0; c < dim; ++c)
                for (int d = 0; d < dim; ++d) J0[c][d] += X0[c * nk + a] * dWq[a * dim + d];
            double adj0[3][3], J0inv[3][3];
            const double det0 = det_d(dim, J0);
            adj_d(dim, J0, adj0);
            for (int c = 0; c < dim; ++c)
              for (int d = 0; d < dim; ++d) J0inv[c][d] = adj0[c][d] / det0;
            double Jpi[3][3];
            for (int c = 0; c < dim; ++c)
              for (int f = 0; f < dim; ++f) {
                double s = 0.0;
                for (int d = 0; d < dim; ++d) s += J[c][d] * J0inv[d][f];
                Jpi[c][f] = s;
              }
            double ls = 0.0;
            for (int c = 0; c < dim; ++c) {
              double s = 0.0;
              for (int f = 0; f < dim; ++f) s += Jpi[c][f] * vec[f * dim + 0];
              ls += s * s;
            }
            const double ell = h0 * sqrt(ls);
            const double lmin = lam[0];
            mu = q_quad * rho * ell * ell * fabs(lmin);
            mu += q_lin * rho * ell * cs * psi0 * (1.0 - smooth_step01(lmin - 2.0 * eps_sw, eps_sw));
            for (int c = 0; c < dim; ++c)
              for (int f = 0; f < dim; ++f) sigma[c][f] += mu * eps[c * dim + f];
          }
          /* step 4 (time step at the point): h_min = sigma_min(J)/k */
          {
            double Jf[9];
            for (int c = 0; c < dim; ++c)
              for (int d = 0; d < dim; ++d) Jf[c * dim + d] = J[c][d];
            const double hmin = oracle_sigma_min(dim, Jf) / (double)k;
            const double inv = cs / hmin + 2.5 * mu / rho / hmin / hmin;
            if (inv > 0.0) {
              const double dtq = cfl / inv;
              if (dtq < dtz) dtz = dtq;
            } else {
              dg[D_NOINV] += 1.0;
            }
          }
          /* step 4 (force): S = alpha sigma adj(J)^T; (A_z)_{(c,a),q} = sum_d S_cd dW_a/dxi_d  (eq 5) */
          double S[3][3];
          for (int c = 0; c < dim; ++c)
            for (int d = 0; d < dim; ++d) {
              double s = 0.0;
              for (int f = 0; f < dim; ++f) s += sigma[c][f] * adjJ[d][f];
              S[c][d] = T.alpha[q] * s;
            }
          for (int c = 0; c < dim; ++c)
            for (int a = 0; a < nk; ++a) {
              double s = 0.0;
              for (int d = 0; d < dim; ++d) s += S[c][d] * dWq[a * dim + d];
              Acol[c * nk + a] = s;
            }
          if (Fz) {
            /* F_z = A_z B^T (eq 5-6, kernel 7): accumulate column q's outer product */
            for (int i = 0; i < dk; ++i)
              for (int j = 0; j < nt; ++j) Fz[(size_t)i * nt + j] += Acol[i] * phq[j];
          } else {
            /* F_z 1 = A_z (B^T 1);  F_z^T V = B (A_z^T V) */
            double b1 = 0.0;
            for (int j = 0; j < nt; ++j) b1 += phq[j];
            for (int i = 0; i < dk; ++i) Fz1[i] += Acol[i] * b1;
            double u = 0.0;
            for (int i = 0; i < dk; ++i) u += Acol[i] * Vz[i];
            for (int j = 0; j < nt; ++j) FTv[j] += phq[j] * u;
          }
        }
        if (Fz) {
          /* kernel 8 (F.1) and kernel 10 (F^T v) on the formed F_z */
          for (int i = 0; i < dk; ++i) {
            double s = 0.0;
            for (int j = 0; j < nt; ++j) s += Fz[(size_t)i * nt + j];
            Fz1[i] = s;
          }
          for (int j = 0; j < nt; ++j) {
            double s = 0.0;
            for (int i = 0; i < dk; ++i) s += Fz[(size_t)i * nt + j] * Vz[i];
            FTv[j] = s;
          }
          memcpy(out_Fz + (size_t)s * dk * nt, Fz, sizeof(double) * (size_t)dk * nt);
        }
        if (bad) dtz = 0.0;
        dt_all[s] = dtz;
        if (out_FTv) memcpy(out_FTv + (size_t)s * nt, FTv, sizeof(double) * nt);
      }
    }
    free(X); free(Vz); free(X0); free(Acol); free(FTv); free(Fz);
  }
  if (failed) { tables_free(&T); free(Fz1_all); free(dt_all); free(dg_all); return -1; }
  /* step 5: serial assembly in ascending zone id; min dt; diagnostics */
  if (out_F1) {
    for (int64_t i = 0; i < (int64_t)dim * nnodes; ++i) out_F1[i] = 0.0;
    for (int64_t s = 0; s < nsub; ++s) {
      const int64_t z = zone_list ? zone_list[s] : s;
      for (int c = 0; c < dim; ++c)
        for (int a = 0; a < nk; ++a) out_F1[c * nnodes + zone_nodes[z * nk + a]] += Fz1_all[(size_t)s * dk + c * nk + a];
    }
  }
  if (out_Fz1) memcpy(out_Fz1, Fz1_all, sizeof(double) * (size_t)nsub * dk);
  if (out_dtz) memcpy(out_dtz, dt_all, sizeof(double) * (size_t)nsub);
  double dtmin = INFINITY;
  for (int64_t s = 0; s < nsub; ++s)
    if (dt_all[s] < dtmin) dtmin = dt_all[s];
  if (out_dt_min) *out_dt_min = dtmin;
  if (diag) {
    diag[D_MINDET] = INFINITY; diag[D_MINGAP] = INFINITY; diag[D_MINSW] = INFINITY;
    diag[D_NOINV] = 0.0; diag[D_NBAD] = 0.0;
    for (int64_t s = 0; s < nsub; ++s) {
      const double *dg = dg_all + (size_t)s * D_COUNT;
      if (dg[D_MINDET] < diag[D_MINDET]) diag[D_MINDET] = dg[D_MINDET];
      if (dg[D_MINGAP] < diag[D_MINGAP]) diag[D_MINGAP] = dg[D_MINGAP];
      if (dg[D_MINSW] < diag[D_MINSW]) diag[D_MINSW] = dg[D_MINSW];
      diag[D_NOINV] += dg[D_NOINV];
      diag[D_NBAD] += dg[D_NBAD];
    }
  }
  tables_free(&T);
  free(Fz1_all); free(dt_all); free(dg_all);
  return 0;
}

int oracle_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}
