/*
 * oracle/mako_oracle.c -- CPU ORACLE for the Mako direct-SCF J/K hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_sc_han0jlacz0025_b200/) never links, imports or executes it, and it
 * shares no code, header, table or constant generator with the CUDA path.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, Han et al. SC'25):
 *   - ERIs (ab|cd) = double integral phi_a phi_b r12^-1 phi_c phi_d      PAPER.md:L106-L109 (S2.1, Eq. 1)
 *     over contracted Gaussians phi = sum_i c_i varphi_i                  PAPER.md:L111-L115 (Eq. 2)
 *     grouped into shells of 2l+1 spherical functions
 *   - J_{mn} = sum_{ls} (mn|ls) D_{ls},  K_{ml} = sum_{ns} (mn|ls) D_{ns}  (BASELINE.json north_star)
 *   - Schwarz screening Q_ab = sqrt(max |(ab|ab)|), keep iff Q_ab Q_cd >= tau
 *     (reading: DESIGN.md "Readings" R6)
 *   - one-electron S, T, V for the RHF energy checks (support only).
 *
 * Deliberately a DIFFERENT algorithm from the GPU path (which is McMurchie-Davidson,
 * PAPER.md:L164-L190 Eq. 4-7): here primitive ERIs come from the Obara-Saika vertical
 * recurrence (PAPER.md:L118 ref [118]) followed by the Head-Gordon-Pople horizontal
 * recurrence (ref [58]); the Boys function is evaluated in long double by its power
 * series / erf closed form (PAPER.md:L177 names F_m; accuracy reading R1 in DESIGN.md);
 * the Cartesian->spherical map is built from the explicit Schlegel-Frisch / Helgaker
 * binomial formula for real solid harmonics (GPU side uses a recurrence).
 *
 * Conventions (identical contract to include/mako.h, derived independently):
 *   Cartesian order within a shell: lx descending, then ly descending (xx,xy,xz,yy,yz,zz).
 *   Spherical order: p = (x,y,z); l>=2: m = -l..l, real solid harmonics with positive
 *   leading terms (PySCF-compatible).  Cartesian functions are normalised so that the
 *   x^l component has unit norm.
 *
 * Parity status: every function here is pinned by tests/test_oracle_*.py against
 * closed forms, mpmath, invariants and published energies.
 */
#include <math.h>
#include <stdlib.h>
#include <string.h>
#include <stdint.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ORC_LMAX 4            /* shells up to g */
#define ORC_LTOT (4 * ORC_LMAX)

/* ------------------------------------------------------------------ */
/* small helpers                                                       */
/* ------------------------------------------------------------------ */
static int ncart(int l) { return (l + 1) * (l + 2) / 2; }
static int nsph(int l) { return 2 * l + 1; }
static int nfun(int l, int pure) { return pure ? nsph(l) : ncart(l); }
/* number of Cartesian tuples with total degree <= L */
static int ncum(int L) { return (L + 1) * (L + 2) * (L + 3) / 6; }
/* index of Cartesian tuple (x,y,z) within its shell (lx descending, ly descending) */
static int cidx(int x, int y, int z) {
  int l = x + y + z;
  return (l - x) * (l - x + 1) / 2 + (l - x - y);
}
/* global index over all tuples of degree <= L: offset of degree l + in-shell index */
static int gidx(int x, int y, int z) {
  int l = x + y + z;
  return (l == 0 ? 0 : ncum(l - 1)) + cidx(x, y, z);
}
/* enumerate tuples of degree l in order; fills xyz[3*ncart(l)] */
static void cart_list(int l, int* xyz) {
  int n = 0;
  for (int x = l; x >= 0; --x)
    for (int y = l - x; y >= 0; --y) {
      xyz[3 * n] = x; xyz[3 * n + 1] = y; xyz[3 * n + 2] = l - x - y; ++n;
    }
}
static double dfact(int n) { /* (n)!! with (-1)!! = 1 */
  double r = 1.0;
  for (int k = n; k > 1; k -= 2) r *= k;
  return r;
}
static double fact(int n) { double r = 1; for (int k = 2; k <= n; ++k) r *= k; return r; }
static double binom(int n, int k) {
  if (k < 0 || k > n) return 0.0;
  return fact(n) / (fact(k) * fact(n - k));
}

/* ------------------------------------------------------------------ */
/* Boys function F_m(T) = int_0^1 t^{2m} exp(-T t^2) dt  */
/* long double: series for T < 30, erf closed form + upward recursion above. */
/* ------------------------------------------------------------------ */
static void boys_ld(int mmax, long double T, long double* F) {
  if (T < 30.0L) {
    /* F_mmax by its power series, then the exact downward recursion
       F_m = (2T F_{m+1} + e^{-T}) / (2m+1). */
    long double eT = expl(-T);
    long double term = 1.0L / (2 * mmax + 1), sum = term;
    for (int k = 1; k < 2000; ++k) {
      term *= 2.0L * T / (2 * mmax + 2 * k + 1);
      sum += term;
      if (term < 1e-22L * sum) break;
    }
    F[mmax] = eT * sum;
    for (int m = mmax - 1; m >= 0; --m) F[m] = (2.0L * T * F[m + 1] + eT) / (2 * m + 1);
  } else {
    long double eT = expl(-T);
    long double sT = sqrtl(T);
    F[0] = 0.5L * sqrtl(3.14159265358979323846264338327950288L / T) * erfl(sT);
    for (int m = 0; m < mmax; ++m) F[m + 1] = ((2 * m + 1) * F[m] - eT) / (2.0L * T);
  }
}

int orc_boys(int mmax, double T, double* out) {
  if (mmax < 0 || mmax > 64 || !(T >= 0)) return 1;
  long double F[65];
  boys_ld(mmax, (long double)T, F);
  for (int m = 0; m <= mmax; ++m) out[m] = (double)F[m];
  return 0;
}

/* ------------------------------------------------------------------ */
/* Cartesian -> spherical: Helgaker/Schlegel-Frisch explicit formula     */
/* S_lm ~ sum_{tuv} C^{lm}_{tuv} x^{2t+|m|-2(u+v)} y^{2(u+v)} z^{l-2t-|m|}  */
/* C = (-1)^{t+v-vm} (1/4)^t binom(l,t) binom(l-t,|m|+t) binom(t,u) binom(|m|,2v) */
/* then normalised in the metric of our Cartesian functions.            */
/* ------------------------------------------------------------------ */
static double sph_tab[ORC_LMAX + 1][2 * ORC_LMAX + 1][(ORC_LMAX + 1) * (ORC_LMAX + 2) / 2];
static int sph_ready = 0;

/* overlap between two normalised Cartesian functions of the same shell (same exponent, center) */
static double cart_metric(int l, const int* a, const int* b) {
  int sx = a[0] + b[0], sy = a[1] + b[1], sz = a[2] + b[2];
  if ((sx | sy | sz) & 1) return 0.0;
  return dfact(sx - 1) * dfact(sy - 1) * dfact(sz - 1) / dfact(2 * l - 1);
}

static void build_sph(void) {
  if (sph_ready) return;
  for (int l = 0; l <= ORC_LMAX; ++l) {
    int xyz[3 * 15];
    cart_list(l, xyz);
    int nc = ncart(l);
    for (int m = -l; m <= l; ++m) {
      double c[15] = {0};
      int am = abs(m);
      /* 2*vm: 0 for m>=0, 1 for m<0; v = vm + k, 2v = 2vm + 2k */
      int twovm = (m < 0) ? 1 : 0;
      for (int t = 0; t <= (l - am) / 2; ++t)
        for (int u = 0; u <= t; ++u)
          for (int twov = twovm; twov <= am; twov += 2) {
            /* sign (-1)^{t + v - vm} with v - vm = (twov - twovm)/2 */
            int sgn_exp = t + (twov - twovm) / 2;
            double coef = ((sgn_exp & 1) ? -1.0 : 1.0) * pow(0.25, t) * binom(l, t) *
                          binom(l - t, am + t) * binom(t, u) * binom(am, twov);
            int px = 2 * t + am - 2 * u - twov;   /* 2t+|m|-2(u+v) */
            int py = 2 * u + twov;                /* 2(u+v) */
            int pz = l - 2 * t - am;
            if (px < 0 || py < 0 || pz < 0) continue;
            c[cidx(px, py, pz)] += coef;
          }
      double nrm = 0;
      for (int i = 0; i < nc; ++i)
        for (int j = 0; j < nc; ++j) nrm += c[i] * c[j] * cart_metric(l, xyz + 3 * i, xyz + 3 * j);
      nrm = 1.0 / sqrt(nrm);
      /* p shells keep the (x,y,z) order rather than m = -1,0,1 */
      int row = (l == 1) ? (m == 1 ? 0 : (m == -1 ? 1 : 2)) : (m + l);
      for (int i = 0; i < nc; ++i) sph_tab[l][row][i] = c[i] * nrm;
    }
  }
  sph_ready = 1;
}

int orc_sph_coeffs(int l, double* out /* [2l+1][ncart(l)] */) {
  if (l < 0 || l > ORC_LMAX) return 1;
  build_sph();
  for (int i = 0; i < nsph(l); ++i)
    for (int j = 0; j < ncart(l); ++j) out[i * ncart(l) + j] = sph_tab[l][i][j];
  return 0;
}

/* ------------------------------------------------------------------ */
/* Basis description passed on every call (no state).                   */
/* ------------------------------------------------------------------ */
typedef struct {
  int nshell;
  const int* l;
  const int* nprim;
  const double* xyz;   /* [nshell][3] bohr */
  const double* exps;  /* concatenated */
  const double* coefs; /* concatenated, for normalised primitives */
  int pure;
  /* derived */
  int* poff;           /* primitive offset per shell */
  int* aoff;           /* AO offset per shell */
  double* cn;          /* contraction coefficient x primitive normalisation x contraction renorm */
  int nbf;
} basis_t;

static int basis_init(basis_t* B, int nshell, const int* l, const int* nprim, const double* xyz,
                      const double* exps, const double* coefs, int pure) {
  B->nshell = nshell; B->l = l; B->nprim = nprim; B->xyz = xyz; B->exps = exps; B->coefs = coefs; B->pure = pure;
  B->poff = (int*)malloc(sizeof(int) * (nshell + 1));
  B->aoff = (int*)malloc(sizeof(int) * (nshell + 1));
  int np = 0, nb = 0;
  for (int s = 0; s < nshell; ++s) {
    if (l[s] < 0 || l[s] > ORC_LMAX || nprim[s] < 1) return 1;
    B->poff[s] = np; B->aoff[s] = nb;
    np += nprim[s]; nb += nfun(l[s], pure);
  }
  B->poff[nshell] = np; B->aoff[nshell] = nb; B->nbf = nb;
  B->cn = (double*)malloc(sizeof(double) * (np ? np : 1));
  /* primitive normalisation N(a,l) = (2a/pi)^{3/4} (4a)^{l/2} / sqrt((2l-1)!!) (x^l component),
     then renormalise the contraction so <x^l|x^l> = 1. */
  for (int s = 0; s < nshell; ++s) {
    int L = l[s];
    for (int i = 0; i < nprim[s]; ++i) {
      double a = exps[B->poff[s] + i];
      double N = pow(2.0 * a / M_PI, 0.75) * pow(4.0 * a, 0.5 * L) / sqrt(dfact(2 * L - 1));
      B->cn[B->poff[s] + i] = coefs[B->poff[s] + i] * N;
    }
    double S = 0;
    for (int i = 0; i < nprim[s]; ++i)
      for (int j = 0; j < nprim[s]; ++j) {
        double p = exps[B->poff[s] + i] + exps[B->poff[s] + j];
        S += B->cn[B->poff[s] + i] * B->cn[B->poff[s] + j] * dfact(2 * L - 1) / pow(2.0 * p, L) *
             pow(M_PI / p, 1.5);
      }
    for (int i = 0; i < nprim[s]; ++i) B->cn[B->poff[s] + i] /= sqrt(S);
  }
  build_sph();
  return 0;
}
static void basis_free(basis_t* B) { free(B->poff); free(B->aoff); free(B->cn); }

int orc_nbf(int nshell, const int* l, int pure) {
  int n = 0;
  for (int s = 0; s < nshell; ++s) n += nfun(l[s], pure);
  return n;
}

/* ------------------------------------------------------------------ */
/* Head-Gordon-Pople horizontal recurrence on the leading index:          */
/*   (a, b+1_i| = (a+1_i, b| + (A_i - B_i) (a, b|                         */
/* in:  [gidx(e) for |e| <= la+lb][nf]  (only |e| >= la used)              */
/* out: [ncart(la)][ncart(lb)][nf]                                         */
/* ------------------------------------------------------------------ */
/* The ERI pipeline (VRR, HRR, contraction, spherical transform) runs in long double: the HRR's
 * cancellation at l = 4 with diffuse exponents costs ~1e-10 absolute in double (measured as the
 * spread between permuted evaluations of one quartet), the size of the north_star ERI bar
 * (reading R22). */
typedef long double real_t;

static void hrr(int la, int lb, const real_t AB[3], int nf, const real_t* in, real_t* out) {
  int Lab = la + lb;
  if (lb == 0) {
    int xyz[3 * 15 * 2];
    cart_list(la, xyz);
    for (int i = 0; i < ncart(la); ++i)
      memcpy(out + (size_t)i * nf, in + (size_t)gidx(xyz[3 * i], xyz[3 * i + 1], xyz[3 * i + 2]) * nf,
             sizeof(real_t) * nf);
    return;
  }
  /* T_j[e][b] for |b| = j, |e| in [la, Lab - j]; stored as [gidx(e)][cidx(b)][nf] */
  int ne = ncum(Lab);
  real_t* prev = (real_t*)calloc((size_t)ne * 1 * nf, sizeof(real_t));
  memcpy(prev, in, sizeof(real_t) * (size_t)ne * nf);
  int nbprev = 1;
  for (int j = 1; j <= lb; ++j) {
    int nb = ncart(j);
    real_t* cur = (real_t*)calloc((size_t)ne * nb * nf, sizeof(real_t));
    int bl[3 * 45];
    cart_list(j, bl);
    for (int le = la; le <= Lab - j; ++le) {
      int el[3 * 45];
      cart_list(le, el);
      for (int ie = 0; ie < ncart(le); ++ie) {
        int ex = el[3 * ie], ey = el[3 * ie + 1], ez = el[3 * ie + 2];
        for (int ib = 0; ib < nb; ++ib) {
          int b[3] = {bl[3 * ib], bl[3 * ib + 1], bl[3 * ib + 2]};
          int d = (b[0] > 0) ? 0 : (b[1] > 0 ? 1 : 2);
          int bm[3] = {b[0], b[1], b[2]};
          bm[d] -= 1;
          int ep[3] = {ex, ey, ez};
          ep[d] += 1;
          const real_t* t1 = prev + ((size_t)gidx(ep[0], ep[1], ep[2]) * nbprev + cidx(bm[0], bm[1], bm[2])) * nf;
          const real_t* t2 = prev + ((size_t)gidx(ex, ey, ez) * nbprev + cidx(bm[0], bm[1], bm[2])) * nf;
          real_t* o = cur + ((size_t)gidx(ex, ey, ez) * nb + ib) * nf;
          for (int k = 0; k < nf; ++k) o[k] = t1[k] + AB[d] * t2[k];
        }
      }
    }
    free(prev);
    prev = cur;
    nbprev = nb;
  }
  int al[3 * 45];
  cart_list(la, al);
  for (int ia = 0; ia < ncart(la); ++ia)
    for (int ib = 0; ib < ncart(lb); ++ib)
      memcpy(out + ((size_t)ia * ncart(lb) + ib) * nf,
             prev + ((size_t)gidx(al[3 * ia], al[3 * ia + 1], al[3 * ia + 2]) * nbprev + ib) * nf,
             sizeof(real_t) * nf);
  free(prev);
}

/* ------------------------------------------------------------------ */
/* Obara-Saika VRR for one primitive quartet, accumulated (x coef) into   */
/* acc[gidx(e)][gidx(f)] for |e| <= Le, |f| <= Lf  (only m = 0 kept).        */
/* work: (ncum(Le) * ncum(Lf) * (Le+Lf+1)) real_ts                          */
/* ------------------------------------------------------------------ */
static void os_vrr_prim(int Le, int Lf, real_t a, const double* A, real_t b, const double* B, real_t c,
                        const double* C, real_t d, const double* D, real_t coef, real_t* acc, real_t* work) {
  const int L = Le + Lf;
  const int nE = ncum(Le), nF = ncum(Lf), nM = L + 1;
  real_t p = a + b, q = c + d, rho = p * q / (p + q);
  real_t P[3], Q[3], W[3], PA[3], QC[3], WP[3], WQ[3], AB2 = 0, CD2 = 0, PQ2 = 0;
  for (int i = 0; i < 3; ++i) {
    P[i] = (a * A[i] + b * B[i]) / p;
    Q[i] = (c * C[i] + d * D[i]) / q;
    W[i] = (p * P[i] + q * Q[i]) / (p + q);
    PA[i] = P[i] - A[i]; QC[i] = Q[i] - C[i]; WP[i] = W[i] - P[i]; WQ[i] = W[i] - Q[i];
    AB2 += (A[i] - B[i]) * (A[i] - B[i]);
    CD2 += (C[i] - D[i]) * (C[i] - D[i]);
    PQ2 += (P[i] - Q[i]) * (P[i] - Q[i]);
  }
  long double F[ORC_LTOT + 1];
  boys_ld(L, (long double)(rho * PQ2), F);
  real_t pref = 2.0L * powl(3.14159265358979323846264338327950288L, 2.5L) / (p * q * sqrtl(p + q)) *
                expl(-a * b / p * AB2 - c * d / q * CD2);
#define V(ei, fi, m) work[((size_t)(ei) * nF + (fi)) * nM + (m)]
  for (int m = 0; m <= L; ++m) V(0, 0, m) = pref * F[m];
  /* build e (f = 0) */
  for (int le = 1; le <= Le; ++le) {
    int el[3 * 91];
    cart_list(le, el);
    for (int ie = 0; ie < ncart(le); ++ie) {
      int e[3] = {el[3 * ie], el[3 * ie + 1], el[3 * ie + 2]};
      int i = (e[0] > 0) ? 0 : (e[1] > 0 ? 1 : 2);
      int e1[3] = {e[0], e[1], e[2]}; e1[i] -= 1;           /* e - 1_i */
      int n1 = e1[i];                                         /* (e-1_i)_i */
      int g = gidx(e[0], e[1], e[2]), g1 = gidx(e1[0], e1[1], e1[2]);
      int g2 = -1;
      if (n1 > 0) { int e2[3] = {e1[0], e1[1], e1[2]}; e2[i] -= 1; g2 = gidx(e2[0], e2[1], e2[2]); }
      for (int m = 0; m <= L - le; ++m) {
        real_t v = PA[i] * V(g1, 0, m) + WP[i] * V(g1, 0, m + 1);
        if (n1 > 0) v += n1 / (2.0 * p) * (V(g2, 0, m) - rho / p * V(g2, 0, m + 1));
        V(g, 0, m) = v;
      }
    }
  }
  /* build f for every e */
  for (int lf = 1; lf <= Lf; ++lf) {
    int fl[3 * 91];
    cart_list(lf, fl);
    for (int jf = 0; jf < ncart(lf); ++jf) {
      int f[3] = {fl[3 * jf], fl[3 * jf + 1], fl[3 * jf + 2]};
      int i = (f[0] > 0) ? 0 : (f[1] > 0 ? 1 : 2);
      int f1[3] = {f[0], f[1], f[2]}; f1[i] -= 1;
      int n1 = f1[i];
      int h = gidx(f[0], f[1], f[2]), h1 = gidx(f1[0], f1[1], f1[2]);
      int h2 = -1;
      if (n1 > 0) { int f2[3] = {f1[0], f1[1], f1[2]}; f2[i] -= 1; h2 = gidx(f2[0], f2[1], f2[2]); }
      for (int le = 0; le <= Le; ++le) {
        int el[3 * 91];
        cart_list(le, el);
        for (int ie = 0; ie < ncart(le); ++ie) {
          int e[3] = {el[3 * ie], el[3 * ie + 1], el[3 * ie + 2]};
          int g = gidx(e[0], e[1], e[2]);
          int ge = -1;
          if (e[i] > 0) { int em[3] = {e[0], e[1], e[2]}; em[i] -= 1; ge = gidx(em[0], em[1], em[2]); }
          for (int m = 0; m <= L - le - lf; ++m) {
            real_t v = QC[i] * V(g, h1, m) + WQ[i] * V(g, h1, m + 1);
            if (n1 > 0) v += n1 / (2.0 * q) * (V(g, h2, m) - rho / q * V(g, h2, m + 1));
            if (e[i] > 0) v += e[i] / (2.0 * (p + q)) * V(ge, h1, m + 1);
            V(g, h, m) = v;
          }
        }
      }
    }
  }
  for (int g = 0; g < nE; ++g)
    for (int h = 0; h < nF; ++h) acc[(size_t)g * nF + h] += coef * V(g, h, 0);
#undef V
}

/* Contracted shell-quartet block (ab|cd) as [na][nb][nc][nd] (pure or Cartesian). */
static void eri_block(const basis_t* B, int sa, int sb, int sc, int sd, double* out) {
  int la = B->l[sa], lb = B->l[sb], lc = B->l[sc], ld = B->l[sd];
  int Le = la + lb, Lf = lc + ld;
  int nE = ncum(Le), nF = ncum(Lf);
  const double *A = B->xyz + 3 * sa, *Bc = B->xyz + 3 * sb, *C = B->xyz + 3 * sc, *D = B->xyz + 3 * sd;
  real_t* acc = (real_t*)calloc((size_t)nE * nF, sizeof(real_t));
  real_t* work = (real_t*)malloc(sizeof(real_t) * (size_t)nE * nF * (Le + Lf + 1));
  for (int i = 0; i < B->nprim[sa]; ++i)
    for (int j = 0; j < B->nprim[sb]; ++j)
      for (int k = 0; k < B->nprim[sc]; ++k)
        for (int m = 0; m < B->nprim[sd]; ++m) {
          int pi = B->poff[sa] + i, pj = B->poff[sb] + j, pk = B->poff[sc] + k, pm = B->poff[sd] + m;
          real_t coef = (real_t)B->cn[pi] * B->cn[pj] * B->cn[pk] * B->cn[pm];
          os_vrr_prim(Le, Lf, B->exps[pi], A, B->exps[pj], Bc, B->exps[pk], C, B->exps[pm], D, coef, acc, work);
        }
  free(work);
  /* bra HRR: [e][f] -> [a][b][f] */
  real_t AB[3] = {A[0] - Bc[0], A[1] - Bc[1], A[2] - Bc[2]};
  real_t CD[3] = {C[0] - D[0], C[1] - D[1], C[2] - D[2]};
  int nca = ncart(la), ncb = ncart(lb), ncc = ncart(lc), ncd = ncart(ld);
  real_t* t1 = (real_t*)malloc(sizeof(real_t) * (size_t)nca * ncb * nF);
  hrr(la, lb, AB, nF, acc, t1);
  /* transpose to [f][ab] for the ket HRR */
  int nab = nca * ncb;
  real_t* t2 = (real_t*)malloc(sizeof(real_t) * (size_t)nF * nab);
  for (int x = 0; x < nab; ++x)
    for (int h = 0; h < nF; ++h) t2[(size_t)h * nab + x] = t1[(size_t)x * nF + h];
  real_t* t3 = (real_t*)malloc(sizeof(real_t) * (size_t)ncc * ncd * nab);
  hrr(lc, ld, CD, nab, t2, t3);
  /* cart[a][b][c][d] */
  real_t* cart = (real_t*)malloc(sizeof(real_t) * (size_t)nab * ncc * ncd);
  for (int x = 0; x < nab; ++x)
    for (int y = 0; y < ncc * ncd; ++y) cart[(size_t)x * ncc * ncd + y] = t3[(size_t)y * nab + x];
  free(acc); free(t1); free(t2); free(t3);
  if (!B->pure) {
    for (size_t x = 0; x < (size_t)nab * ncc * ncd; ++x) out[x] = (double)cart[x];
    free(cart);
    return;
  }
  /* spherical transform index by index */
  int ls[4] = {la, lb, lc, ld};
  int nin[4] = {nca, ncb, ncc, ncd};
  real_t* cur = cart;
  int dims[4] = {nca, ncb, ncc, ncd};
  for (int ax = 0; ax < 4; ++ax) {
    int no = nsph(ls[ax]);
    int pre = 1, post = 1;
    for (int k = 0; k < ax; ++k) pre *= dims[k];
    for (int k = ax + 1; k < 4; ++k) post *= dims[k];
    real_t* nxt = (real_t*)calloc((size_t)pre * no * post, sizeof(real_t));
    for (int x = 0; x < pre; ++x)
      for (int o = 0; o < no; ++o)
        for (int i = 0; i < nin[ax]; ++i) {
          real_t cf = sph_tab[ls[ax]][o][i];
          if (cf == 0.0) continue;
          const real_t* src = cur + ((size_t)x * nin[ax] + i) * post;
          real_t* dst = nxt + ((size_t)x * no + o) * post;
          for (int y = 0; y < post; ++y) dst[y] += cf * src[y];
        }
    free(cur);
    cur = nxt;
    dims[ax] = no;
  }
  for (size_t x = 0; x < (size_t)dims[0] * dims[1] * dims[2] * dims[3]; ++x) out[x] = (double)cur[x];
  free(cur);
}

#define BASIS_ARGS int nshell, const int *l, const int *nprim, const double *xyz, const double *exps, \
                   const double *coefs, int pure
#define BASIS_INIT(B)                                                    \
  basis_t B;                                                             \
  if (basis_init(&B, nshell, l, nprim, xyz, exps, coefs, pure)) { basis_free(&B); return 2; }

/* one shell quartet block [na][nb][nc][nd] */
int orc_eri_quartet(BASIS_ARGS, int a, int b, int c, int d, double* out) {
  BASIS_INIT(B);
  if (a < 0 || b < 0 || c < 0 || d < 0 || a >= nshell || b >= nshell || c >= nshell || d >= nshell) {
    basis_free(&B);
    return 1;
  }
  eri_block(&B, a, b, c, d, out);
  basis_free(&B);
  return 0;
}

/* full ERI tensor [nbf]^4 (brute force, no symmetry used; tiny bases only) */
int orc_eri_full(BASIS_ARGS, double* out) {
  BASIS_INIT(B);
  int N = B.nbf;
#pragma omp parallel for schedule(dynamic) collapse(2)
  for (int a = 0; a < nshell; ++a)
    for (int b = 0; b < nshell; ++b) {
      double* blk = (double*)malloc(sizeof(double) * 2401 * 2401 / 49);
      for (int c = 0; c < nshell; ++c)
        for (int d = 0; d < nshell; ++d) {
          int na = nfun(l[a], pure), nb = nfun(l[b], pure), nc = nfun(l[c], pure), nd = nfun(l[d], pure);
          eri_block(&B, a, b, c, d, blk);
          for (int i = 0; i < na; ++i)
            for (int j = 0; j < nb; ++j)
              for (int k = 0; k < nc; ++k)
                for (int m = 0; m < nd; ++m)
                  out[(((size_t)(B.aoff[a] + i) * N + B.aoff[b] + j) * N + B.aoff[c] + k) * N + B.aoff[d] + m] =
                      blk[((i * nb + j) * nc + k) * nd + m];
        }
      free(blk);
    }
  basis_free(&B);
  return 0;
}

/* Schwarz factors Q[a*nshell+b] = sqrt(max_{mu in a, nu in b} |(mu nu|mu nu)|) */
int orc_schwarz(BASIS_ARGS, double* Q) {
  BASIS_INIT(B);
#pragma omp parallel for schedule(dynamic)
  for (int a = 0; a < nshell; ++a) {
    double* blk = (double*)malloc(sizeof(double) * 50625);
    for (int b = 0; b <= a; ++b) {
      int na = nfun(l[a], pure), nb = nfun(l[b], pure);
      eri_block(&B, a, b, a, b, blk);
      double mx = 0;
      for (int i = 0; i < na; ++i)
        for (int j = 0; j < nb; ++j) {
          double v = fabs(blk[((i * nb + j) * na + i) * nb + j]);
          if (v > mx) mx = v;
        }
      Q[a * nshell + b] = Q[b * nshell + a] = sqrt(mx);
    }
    free(blk);
  }
  basis_free(&B);
  return 0;
}

/* Add the contributions of one canonical quartet block (with degeneracy factor deg)
   to the non-symmetrised accumulators Jacc/Kacc (J = Jacc + Jacc^T, K = Kacc + Kacc^T).
   The 8 index permutations of (ab|cd) each add J_{mn} += (mn|ls) D_ls and
   K_{ml} += (mn|ls) D_ns; for symmetric D the 8 collapse to the 6 "forward" updates below. */
static void digest(const basis_t* B, int a, int b, int c, int d, const double* blk, double deg, const double* Dm,
                   double* J, double* K) {
  int N = B->nbf;
  int na = nfun(B->l[a], B->pure), nb = nfun(B->l[b], B->pure), nc = nfun(B->l[c], B->pure),
      nd = nfun(B->l[d], B->pure);
  int oa = B->aoff[a], ob = B->aoff[b], oc = B->aoff[c], od = B->aoff[d];
  for (int i = 0; i < na; ++i)
    for (int j = 0; j < nb; ++j)
      for (int k = 0; k < nc; ++k)
        for (int m = 0; m < nd; ++m) {
          double v = deg * blk[((i * nb + j) * nc + k) * nd + m];
          int I = oa + i, Jx = ob + j, Kx = oc + k, M = od + m;
          J[(size_t)I * N + Jx] += 2.0 * v * Dm[(size_t)Kx * N + M];
          J[(size_t)Kx * N + M] += 2.0 * v * Dm[(size_t)I * N + Jx];
          K[(size_t)I * N + Kx] += v * Dm[(size_t)Jx * N + M];
          K[(size_t)Jx * N + Kx] += v * Dm[(size_t)I * N + M];
          K[(size_t)I * N + M] += v * Dm[(size_t)Jx * N + Kx];
          K[(size_t)Jx * N + M] += v * Dm[(size_t)I * N + Kx];
        }
}

/* Screened J/K over canonical shell quartets (a>=b, c>=d, ab>=cd); keep iff Q_ab Q_cd >= tau.
   shard/nshards: only canonical bra pairs with (pair_index % nshards == shard) are evaluated
   (an oracle-side sample; the GPU library's own shard partition is not replicated here).
   Qin: optional precomputed Schwarz table (orc_schwarz), NULL to compute it here.
   J, K: [nbf][nbf] outputs (overwritten), final symmetrised values. */
static int jk_impl(BASIS_ARGS, const double* Dm, double tau, double tau_dw, long long shard, long long nshards,
                   int qsample, const double* Qin, double* Jout, double* Kout);

int orc_jk(BASIS_ARGS, const double* Dm, double tau, int shard, int nshards, const double* Qin, double* Jout,
           double* Kout) {
  return jk_impl(nshell, l, nprim, xyz, exps, coefs, pure, Dm, tau, -1.0, shard, nshards, 0, Qin, Jout, Kout);
}

/* Quartet-level sample (for timing the oracle on a bounded part of a large build; bench.py cpu_baseline):
   as orc_jk, but the canonical quartet (P, R), R <= P (pair index P = a(a+1)/2 + b), is evaluated iff
   (P(P+1)/2 + R) % nshards == shard.  Every bra pair and every class is sampled uniformly, so the work
   of one shard is 1/nshards of the build with a small spread; the shards sum to orc_jk (same J/K). */
int orc_jk_qsample(BASIS_ARGS, const double* Dm, double tau, long long shard, long long nshards, const double* Qin,
                   double* Jout, double* Kout) {
  return jk_impl(nshell, l, nprim, xyz, exps, coefs, pure, Dm, tau, -1.0, shard, nshards, 1, Qin, Jout, Kout);
}

/* Density-weighted screening ("density-weighted Schwarz"; reading R17):
   as orc_jk, and a quartet is kept only if also Q_ab Q_cd Dmax >= tau_dw, where Dmax is the largest
   max|D_mn| over the six shell blocks (ab)(cd)(ac)(ad)(bc)(bd) the quartet is contracted with. */
int orc_jk_dw(BASIS_ARGS, const double* Dm, double tau, double tau_dw, const double* Qin, double* Jout,
              double* Kout) {
  if (!(tau_dw >= 0)) return 1;
  return jk_impl(nshell, l, nprim, xyz, exps, coefs, pure, Dm, tau, tau_dw, 0, 1, 0, Qin, Jout, Kout);
}

static int jk_impl(BASIS_ARGS, const double* Dm, double tau, double tau_dw, long long shard, long long nshards,
                   int qsample, const double* Qin, double* Jout, double* Kout) {
  BASIS_INIT(B);
  if (nshards < 1 || shard < 0 || shard >= nshards || tau < 0) { basis_free(&B); return 1; }
  int N = B.nbf;
  double* Q = (double*)malloc(sizeof(double) * nshell * nshell);
  if (Qin) memcpy(Q, Qin, sizeof(double) * nshell * nshell);
  else {
    basis_free(&B);
    orc_schwarz(nshell, l, nprim, xyz, exps, coefs, pure, Q);
    if (basis_init(&B, nshell, l, nprim, xyz, exps, coefs, pure)) return 2;
  }
  int npair = nshell * (nshell + 1) / 2;
  int* pa = (int*)malloc(sizeof(int) * npair);
  int* pb = (int*)malloc(sizeof(int) * npair);
  for (int a = 0, k = 0; a < nshell; ++a)
    for (int b = 0; b <= a; ++b, ++k) { pa[k] = a; pb[k] = b; }
  memset(Jout, 0, sizeof(double) * (size_t)N * N);
  memset(Kout, 0, sizeof(double) * (size_t)N * N);
  /* shell-block maxima of |D| (density-weighted screening only) */
  double* Dsh = (double*)calloc((size_t)nshell * nshell, sizeof(double));
  if (tau_dw >= 0)
    for (int x = 0; x < nshell; ++x)
      for (int y = 0; y < nshell; ++y) {
        double m = 0.0;
        for (int i = 0; i < B.aoff[x + 1] - B.aoff[x]; ++i)
          for (int j = 0; j < B.aoff[y + 1] - B.aoff[y]; ++j) {
            double v = fabs(Dm[(size_t)(B.aoff[x] + i) * N + B.aoff[y] + j]);
            if (v > m) m = v;
          }
        Dsh[x * nshell + y] = m;
      }
#pragma omp parallel
  {
    double* Jl = (double*)calloc((size_t)N * N, sizeof(double));
    double* Kl = (double*)calloc((size_t)N * N, sizeof(double));
    double* blk = (double*)malloc(sizeof(double) * 81 * 81 * 81 * 81 / 81);
#pragma omp for schedule(dynamic, 1)
    for (int P = 0; P < npair; ++P) {
      if (!qsample && P % nshards != shard) continue;
      int a = pa[P], b = pb[P];
      /* quartet sample: first R with (P(P+1)/2 + R) % nshards == shard, then every nshards-th */
      const long long base = (long long)P * (P + 1) / 2;
      const long long R0 = qsample ? ((shard - base % nshards) % nshards + nshards) % nshards : 0;
      if (R0 > P) continue;  /* no quartet of this bra pair in the sample */
      const int Rstep = qsample ? (int)(nshards < (long long)npair + 1 ? nshards : (long long)npair + 1) : 1;
      for (int R = (int)R0; R <= P; R += Rstep) {
        int c = pa[R], d = pb[R];
        double qq = Q[a * nshell + b] * Q[c * nshell + d];
        if (qq < tau) continue;
        if (tau_dw >= 0) {
          double m = Dsh[a * nshell + b];
          double t[5] = {Dsh[c * nshell + d], Dsh[a * nshell + c], Dsh[a * nshell + d], Dsh[b * nshell + c],
                         Dsh[b * nshell + d]};
          for (int z = 0; z < 5; ++z) if (t[z] > m) m = t[z];
          if (qq * m < tau_dw) continue;
        }
        eri_block(&B, a, b, c, d, blk);
        double deg = 1.0;
        if (a == b) deg *= 0.5;
        if (c == d) deg *= 0.5;
        if (P == R) deg *= 0.5;
        digest(&B, a, b, c, d, blk, deg, Dm, Jl, Kl);
      }
    }
#pragma omp critical
    {
      for (size_t x = 0; x < (size_t)N * N; ++x) { Jout[x] += Jl[x]; Kout[x] += Kl[x]; }
    }
    free(Jl); free(Kl); free(blk);
  }
  /* symmetrise: J = Jacc + Jacc^T, K = Kacc + Kacc^T */
  for (int i = 0; i < N; ++i)
    for (int j = 0; j <= i; ++j) {
      double s = Jout[(size_t)i * N + j] + Jout[(size_t)j * N + i];
      Jout[(size_t)i * N + j] = Jout[(size_t)j * N + i] = s;
      s = Kout[(size_t)i * N + j] + Kout[(size_t)j * N + i];
      Kout[(size_t)i * N + j] = Kout[(size_t)j * N + i] = s;
    }
  free(Q); free(pa); free(pb); free(Dsh);
  basis_free(&B);
  return 0;
}

/* Exact J and K blocks for sampled shell pairs, straight from the definitions
   J_{mn} = sum_{ls} (mn|ls) D_ls (m in x, n in y) and K_{ml} = sum_{ns} (mn|ls) D_ns (m in x, l in y),
   with the same Schwarz rule (quartet (x b|y d) kept iff Q_xb Q_yd >= tau).
   Q: caller-provided Schwarz table [nshell][nshell] (from orc_schwarz), or NULL to compute.
   Jblk/Kblk: concatenated [n_x][n_y] blocks per requested pair. */
int orc_jk_blocks(BASIS_ARGS, const double* Dm, double tau, const double* Qin, int npairs, const int* pairs,
                  double* Jblk, double* Kblk) {
  BASIS_INIT(B);
  int N = B.nbf;
  double* Q = (double*)malloc(sizeof(double) * nshell * nshell);
  if (Qin) memcpy(Q, Qin, sizeof(double) * nshell * nshell);
  else {
    basis_free(&B);
    orc_schwarz(nshell, l, nprim, xyz, exps, coefs, pure, Q);
    if (basis_init(&B, nshell, l, nprim, xyz, exps, coefs, pure)) return 2;
  }
  size_t* boff = (size_t*)malloc(sizeof(size_t) * (npairs + 1));
  boff[0] = 0;
  for (int k = 0; k < npairs; ++k)
    boff[k + 1] = boff[k] + (size_t)nfun(l[pairs[2 * k]], pure) * nfun(l[pairs[2 * k + 1]], pure);
  for (int k = 0; k < npairs; ++k) {
    int x = pairs[2 * k], y = pairs[2 * k + 1];
    int nx = nfun(l[x], pure), ny = nfun(l[y], pure);
    double* Jo = Jblk + boff[k];
    double* Ko = Kblk + boff[k];
    memset(Jo, 0, sizeof(double) * nx * ny);
    memset(Ko, 0, sizeof(double) * nx * ny);
    /* J block: sum over all shells c, d of (x y|c d) D_cd */
#pragma omp parallel
    {
      double* blk = (double*)malloc(sizeof(double) * 81 * 81 * 81);
      double* Jl = (double*)calloc(nx * ny, sizeof(double));
      double* Kl = (double*)calloc(nx * ny, sizeof(double));
#pragma omp for schedule(dynamic, 4)
      for (int c = 0; c < nshell; ++c) {
        for (int d = 0; d < nshell; ++d) {
          int nc = nfun(l[c], pure), nd = nfun(l[d], pure);
          if (Q[x * nshell + y] * Q[c * nshell + d] >= tau) {
            eri_block(&B, x, y, c, d, blk);
            for (int i = 0; i < nx; ++i)
              for (int j = 0; j < ny; ++j) {
                double s = 0;
                for (int kk = 0; kk < nc; ++kk)
                  for (int m = 0; m < nd; ++m)
                    s += blk[((i * ny + j) * nc + kk) * nd + m] * Dm[(size_t)(B.aoff[c] + kk) * N + B.aoff[d] + m];
                Jl[i * ny + j] += s;
              }
          }
          /* K block: here (c, d) play the roles of (b, d) in (x b|y d) */
          if (Q[x * nshell + c] * Q[y * nshell + d] >= tau) {
            eri_block(&B, x, c, y, d, blk);
            for (int i = 0; i < nx; ++i)
              for (int j = 0; j < ny; ++j) {
                double s = 0;
                for (int kk = 0; kk < nc; ++kk)
                  for (int m = 0; m < nd; ++m)
                    s += blk[((i * nc + kk) * ny + j) * nd + m] * Dm[(size_t)(B.aoff[c] + kk) * N + B.aoff[d] + m];
                Kl[i * ny + j] += s;
              }
          }
        }
      }
#pragma omp critical
      for (int i = 0; i < nx * ny; ++i) { Jo[i] += Jl[i]; Ko[i] += Kl[i]; }
      free(blk); free(Jl); free(Kl);
    }
  }
  free(boff); free(Q);
  basis_free(&B);
  return 0;
}

/* ------------------------------------------------------------------ */
/* one-electron integrals (support for the RHF energy pins)              */
/* ------------------------------------------------------------------ */
/* 1D Obara-Saika overlap table s[i][j], i <= imax, j <= jmax (without the exp prefactor and sqrt(pi/p)) */
static void os_overlap_1d(int imax, int jmax, double PA, double PB, double p, double* s /* [(imax+1)*(jmax+1)] */) {
  int nj = jmax + 1;
  for (int i = 0; i <= imax; ++i)
    for (int j = 0; j <= jmax; ++j) {
      double v;
      if (i == 0 && j == 0) v = 1.0;
      else if (i > 0) {
        v = PA * s[(i - 1) * nj + j];
        if (i > 1) v += (i - 1) / (2 * p) * s[(i - 2) * nj + j];
        if (j > 0) v += j / (2 * p) * s[(i - 1) * nj + j - 1];
      } else {
        v = PB * s[i * nj + j - 1];
        if (j > 1) v += (j - 1) / (2 * p) * s[i * nj + j - 2];
      }
      s[i * nj + j] = v;
    }
}

/* Cartesian primitive overlap and kinetic for tuples ea, eb */
static void prim_ST(double a, const double* A, const int* ea, double b, const double* Bc, const int* eb, double* S,
                    double* T) {
  double p = a + b, mu = a * b / p;
  double sx[3][(ORC_LMAX + 1) * (ORC_LMAX + 3)];
  int jm = ORC_LMAX + 2;
  double ovl[3], kin[3];
  double pre = pow(M_PI / p, 1.5);
  double AB2 = 0;
  for (int k = 0; k < 3; ++k) {
    double P = (a * A[k] + b * Bc[k]) / p;
    AB2 += (A[k] - Bc[k]) * (A[k] - Bc[k]);
    os_overlap_1d(ORC_LMAX, jm, P - A[k], P - Bc[k], p, sx[k]);
    int i = ea[k], j = eb[k];
    ovl[k] = sx[k][i * (jm + 1) + j];
    double t = -2.0 * b * b * sx[k][i * (jm + 1) + j + 2] + b * (2 * j + 1) * sx[k][i * (jm + 1) + j];
    if (j >= 2) t += -0.5 * j * (j - 1) * sx[k][i * (jm + 1) + j - 2];
    kin[k] = t;
  }
  double E = exp(-mu * AB2) * pre;
  *S = E * ovl[0] * ovl[1] * ovl[2];
  *T = E * (kin[0] * ovl[1] * ovl[2] + ovl[0] * kin[1] * ovl[2] + ovl[0] * ovl[1] * kin[2]);
}

/* nuclear attraction (a| -Z/|r-C| |b) primitive, Obara-Saika VRR over tuples up to la+lb then HRR */
static void prim_V_acc(int la, int lb, double a, const double* A, double b, const double* Bc, int natm, const double* Z,
                       const double* Cxyz, double coef, double* acc /* [gidx(e)] for |e|<=la+lb */) {
  int L = la + lb, nE = ncum(L);
  double p = a + b, P[3], PA[3], AB2 = 0;
  for (int k = 0; k < 3; ++k) {
    P[k] = (a * A[k] + b * Bc[k]) / p; PA[k] = P[k] - A[k];
    AB2 += (A[k] - Bc[k]) * (A[k] - Bc[k]);
  }
  double* V = (double*)malloc(sizeof(double) * nE * (L + 1));
  for (int n = 0; n < natm; ++n) {
    double PC[3], PC2 = 0;
    for (int k = 0; k < 3; ++k) { PC[k] = P[k] - Cxyz[3 * n + k]; PC2 += PC[k] * PC[k]; }
    long double F[ORC_LTOT + 1];
    boys_ld(L, (long double)(p * PC2), F);
    double pre = -Z[n] * 2.0 * M_PI / p * exp(-a * b / p * AB2);
    for (int m = 0; m <= L; ++m) V[m] = pre * (double)F[m];
    for (int le = 1; le <= L; ++le) {
      int el[3 * 91];
      cart_list(le, el);
      for (int ie = 0; ie < ncart(le); ++ie) {
        int e[3] = {el[3 * ie], el[3 * ie + 1], el[3 * ie + 2]};
        int i = (e[0] > 0) ? 0 : (e[1] > 0 ? 1 : 2);
        int e1[3] = {e[0], e[1], e[2]}; e1[i] -= 1;
        int n1 = e1[i];
        int g = gidx(e[0], e[1], e[2]), g1 = gidx(e1[0], e1[1], e1[2]), g2 = -1;
        if (n1 > 0) { int e2[3] = {e1[0], e1[1], e1[2]}; e2[i] -= 1; g2 = gidx(e2[0], e2[1], e2[2]); }
        for (int m = 0; m <= L - le; ++m) {
          double v = PA[i] * V[g1 * (L + 1) + m] - PC[i] * V[g1 * (L + 1) + m + 1];
          if (n1 > 0) v += n1 / (2.0 * p) * (V[g2 * (L + 1) + m] - V[g2 * (L + 1) + m + 1]);
          V[g * (L + 1) + m] = v;
        }
      }
    }
    for (int g = 0; g < nE; ++g) acc[g] += coef * V[g * (L + 1)];
  }
  free(V);
}

static void sph_2idx(const basis_t* B, int la, int lb, const double* cart, double* out) {
  int nca = ncart(la), ncb = ncart(lb);
  if (!B->pure) { memcpy(out, cart, sizeof(double) * nca * ncb); return; }
  int nsa = nsph(la), nsb = nsph(lb);
  for (int i = 0; i < nsa; ++i)
    for (int j = 0; j < nsb; ++j) {
      double s = 0;
      for (int x = 0; x < nca; ++x)
        for (int y = 0; y < ncb; ++y) s += sph_tab[la][i][x] * sph_tab[lb][j][y] * cart[x * ncb + y];
      out[i * nsb + j] = s;
    }
}

/* S, T, V [nbf][nbf]; atoms: natm, Z (as double charges), xyz [natm][3] */
int orc_one_electron(BASIS_ARGS, int natm, const double* Z, const double* axyz, double* S, double* T, double* Vout) {
  BASIS_INIT(B);
  int N = B.nbf;
  for (int sa = 0; sa < nshell; ++sa)
    for (int sb = 0; sb < nshell; ++sb) {
      int la = l[sa], lb = l[sb], nca = ncart(la), ncb = ncart(lb);
      int al[3 * 15], bl[3 * 15];
      cart_list(la, al); cart_list(lb, bl);
      double cs[225] = {0}, ct[225] = {0}, cv[225] = {0};
      const double *A = xyz + 3 * sa, *Bc = xyz + 3 * sb;
      double* vacc = (double*)calloc(ncum(la + lb), sizeof(double));
      double* vab = (double*)malloc(sizeof(double) * nca * ncb);
      for (int i = 0; i < nprim[sa]; ++i)
        for (int j = 0; j < nprim[sb]; ++j) {
          int pi = B.poff[sa] + i, pj = B.poff[sb] + j;
          double cf = B.cn[pi] * B.cn[pj];
          for (int x = 0; x < nca; ++x)
            for (int y = 0; y < ncb; ++y) {
              double s, t;
              prim_ST(exps[pi], A, al + 3 * x, exps[pj], Bc, bl + 3 * y, &s, &t);
              cs[x * ncb + y] += cf * s;
              ct[x * ncb + y] += cf * t;
            }
          prim_V_acc(la, lb, exps[pi], A, exps[pj], Bc, natm, Z, axyz, cf, vacc);
        }
      real_t ABv[3] = {A[0] - Bc[0], A[1] - Bc[1], A[2] - Bc[2]};
      real_t* vaccl = (real_t*)malloc(sizeof(real_t) * ncum(la + lb));
      real_t* vabl = (real_t*)malloc(sizeof(real_t) * nca * ncb);
      for (int x = 0; x < ncum(la + lb); ++x) vaccl[x] = vacc[x];
      hrr(la, lb, ABv, 1, vaccl, vabl);
      for (int x = 0; x < nca * ncb; ++x) cv[x] = (double)vabl[x];
      free(vacc); free(vab); free(vaccl); free(vabl);
      double os[225], ot[225], ov[225];
      sph_2idx(&B, la, lb, cs, os);
      sph_2idx(&B, la, lb, ct, ot);
      sph_2idx(&B, la, lb, cv, ov);
      int na = nfun(la, pure), nb = nfun(lb, pure);
      for (int i = 0; i < na; ++i)
        for (int j = 0; j < nb; ++j) {
          size_t ix = (size_t)(B.aoff[sa] + i) * N + B.aoff[sb] + j;
          S[ix] = os[i * nb + j]; T[ix] = ot[i * nb + j]; Vout[ix] = ov[i * nb + j];
        }
    }
  basis_free(&B);
  return 0;
}

int orc_num_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}
