"""Independent helpers for the oracle pins: numpy-only closed forms, never the oracle's own code.

GLL nodes/weights here come from numpy's Legendre class (a library routine independent of the
oracle's long-double Newton iteration); exact-rational polynomial algebra uses fractions.Fraction.
"""
from fractions import Fraction
from itertools import product

import numpy as np


def gll01(k):
    """GLL nodes and weights on [0,1] from numpy: w_i = 1 / (k(k+1) P_k(x_i)^2) (halved [-1,1] rule)."""
    leg = np.polynomial.legendre.Legendre.basis(k)
    if k == 1:
        x = np.array([-1.0, 1.0])
    else:
        x = np.concatenate([[-1.0], np.sort(np.real(leg.deriv().roots())), [1.0]])
    w = 2.0 / (k * (k + 1) * leg(x) ** 2)
    return 0.5 * (x + 1.0), 0.5 * w


def nanson_F1(dim, k, A, p):
    """Closed form of F_z.1 for uniform stress -p I on the affine zone x = A xi (+b):
    (F_z 1)_{c,a} = -p sum_d adj(A)_{dc} (delta_{a_d,k} - delta_{a_d,0}) prod_{t != d} w_{a_t}
    (divergence theorem on the reference element; Nanson's formula).  Returns [dim][nk]."""
    _, w = gll01(k)
    adjA = np.linalg.det(A) * np.linalg.inv(A)
    nk = (k + 1) ** dim
    out = np.zeros((dim, nk))
    for a in range(nk):
        ai = [(a // (k + 1) ** t) % (k + 1) for t in range(dim)]
        for c in range(dim):
            s = 0.0
            for d in range(dim):
                jump = (1.0 if ai[d] == k else 0.0) - (1.0 if ai[d] == 0 else 0.0)
                if jump == 0.0:
                    continue
                wt = 1.0
                for t in range(dim):
                    if t != d:
                        wt *= w[ai[t]]
                s += adjA[d, c] * jump * wt
            out[c, a] = -p * s
    return out


# ---------------------------------------------------------------------------------------------
# exact-rational 1-D polynomials (coefficient lists, ascending powers)
# ---------------------------------------------------------------------------------------------

def pmul(a, b):
    out = [Fraction(0)] * (len(a) + len(b) - 1)
    for i, x in enumerate(a):
        for j, y in enumerate(b):
            out[i + j] += x * y
    return out


def pder(a):
    return [a[i] * i for i in range(1, len(a))] or [Fraction(0)]


def pint01(a):
    return sum(c / (i + 1) for i, c in enumerate(a))


def lagrange_polys(nodes):
    polys = []
    for a, xa in enumerate(nodes):
        p = [Fraction(1)]
        for b, xb in enumerate(nodes):
            if b != a:
                p = pmul(p, [-xb / (xa - xb), Fraction(1) / (xa - xb)])
        polys.append(p)
    return polys


def bernstein_polys(m):
    from math import comb
    polys = []
    for j in range(m + 1):
        p = [Fraction(comb(m, j))]
        for _ in range(j):
            p = pmul(p, [Fraction(0), Fraction(1)])
        for _ in range(m - j):
            p = pmul(p, [Fraction(1), Fraction(-1)])
        polys.append(p)
    return polys


def exact_Fz_affine_novisc(dim, k, A, R, gamma, E):
    """Exact (F_z)_{(c,a),j} = int_[0,1]^d -p(xi) sum_d adj(A)_{dc} dW_a/dxi_d phi_j dxi for the affine
    zone x = A xi, viscosity off, p = (gamma-1) (R/det A) e(xi), e = sum_i E_i phi_i (eq 4 with
    sigma = -p I).  A, R, gamma, E must be given as Fractions (exact).  Returns [dim*nk][nt] Fractions."""
    assert k in (1, 2)
    nodes = [Fraction(0), Fraction(1)] if k == 1 else [Fraction(0), Fraction(1, 2), Fraction(1)]
    L = lagrange_polys(nodes)
    dL = [pder(p) for p in L]
    Bp = bernstein_polys(k - 1)
    if dim == 2:
        detA = A[0][0] * A[1][1] - A[0][1] * A[1][0]
        adj = [[A[1][1], -A[0][1]], [-A[1][0], A[0][0]]]
    else:
        # adj(A)_{ij} = cofactor_{ji}
        def cof(i, j):
            r = [x for x in range(3) if x != i]
            c = [x for x in range(3) if x != j]
            m = A[r[0]][c[0]] * A[r[1]][c[1]] - A[r[0]][c[1]] * A[r[1]][c[0]]
            return m if (i + j) % 2 == 0 else -m
        adj = [[cof(j, i) for j in range(3)] for i in range(3)]
        detA = sum(A[0][j] * cof(0, j) for j in range(3))
    rho = R / detA
    coef = -(gamma - 1) * rho
    p1 = k + 1
    nk, nt = p1 ** dim, k ** dim
    # 1-D integrals I[d-flag][a][i][j] = int W_a^(flag) phi_i phi_j
    I = {}
    for flag, WL in (("v", L), ("d", dL)):
        for a in range(p1):
            for i in range(k):
                for j in range(k):
                    I[(flag, a, i, j)] = pint01(pmul(pmul(WL[a], Bp[i]), Bp[j]))
    F = [[Fraction(0)] * nt for _ in range(dim * nk)]
    for c in range(dim):
        for a in range(nk):
            ai = [(a // p1 ** t) % p1 for t in range(dim)]
            for j in range(nt):
                ji = [(j // k ** t) % k for t in range(dim)]
                s = Fraction(0)
                for ii in range(nt):
                    iv = [(ii // k ** t) % k for t in range(dim)]
                    for d in range(dim):
                        if adj[d][c] == 0:
                            continue
                        term = Fraction(1)
                        for t in range(dim):
                            term *= I[("d" if t == d else "v", ai[t], iv[t], ji[t])]
                        s += E[ii] * adj[d][c] * term
                F[c * nk + a][j] = coef * s
    return F
