// basis.cpp -- mako_basis_create and the library's own host-side tables.
//
//  * contracted-shell normalisation (Eq. 2: phi = sum_i c_i varphi_i; the
//    coefficients refer to normalised primitives; the contraction is renormalised so that its
//    x^l component has unit norm -- include/mako.h conventions);
//  * Cartesian -> real-solid-harmonic tables built by the solid-harmonic RECURRENCE
//    (Helgaker, Jorgensen, Olsen, Eqs. 6.4.70-6.4.72), normalised numerically in the metric of
//    the Cartesian functions (a shell holds 2l+1 spherical CGFs);
//  * the Boys-function Taylor-grid table F_m(T_k) (PAPER.md:L173-L177 names F_m and a lookup
//    table; reading R1 fixes the accuracy contract), evaluated by composite
//    Gauss-Legendre quadrature of F_m(T) = int_0^1 t^{2m} exp(-T t^2) dt in long double.
#include <cmath>
#include <cstring>
#include <cuda_runtime.h>

#include "mako_state.h"

namespace mako {

static thread_local std::string g_err;
void set_error(const std::string& msg) { g_err = msg; }
mako_status fail(mako_status st, const std::string& msg) {
  g_err = msg;
  return st;
}
const char* last_error_cstr() { return g_err.c_str(); }

DevBuf::~DevBuf() { release(); }
void DevBuf::release() {
  if (p) cudaFree(p);
  p = nullptr;
  bytes = 0;
}
mako_status DevBuf::alloc(size_t nbytes) {
  release();
  if (nbytes == 0) nbytes = 8;
  cudaError_t e = cudaMalloc(&p, nbytes);
  if (e != cudaSuccess) {
    p = nullptr;
    return fail(e == cudaErrorMemoryAllocation ? MAKO_ERR_OOM : MAKO_ERR_CUDA,
                std::string("cudaMalloc: ") + cudaGetErrorString(e));
  }
  bytes = nbytes;
  return MAKO_OK;
}

static double dfac(int n) {  // n!! with (-1)!! = 1
  double r = 1.0;
  for (; n > 1; n -= 2) r *= n;
  return r;
}

// ---------------------------------------------------------------------------
// real solid harmonics by recurrence, as coefficient vectors over degree-l monomials
// ---------------------------------------------------------------------------
using Poly = std::vector<double>;  // indexed by cart_index within degree l

static Poly mul_axis(const Poly& s, int l, int axis) {  // degree l -> l+1
  Poly r(ncart(l + 1), 0.0);
  for (int x = l; x >= 0; --x)
    for (int y = l - x; y >= 0; --y) {
      int z = l - x - y;
      double c = s[cart_index(x, y, z)];
      if (c == 0.0) continue;
      int e[3] = {x, y, z};
      e[axis] += 1;
      r[cart_index(e[0], e[1], e[2])] += c;
    }
  return r;
}
static Poly mul_r2(const Poly& s, int l) {  // degree l -> l+2
  Poly r(ncart(l + 2), 0.0);
  for (int a = 0; a < 3; ++a) {
    Poly t = mul_axis(mul_axis(s, l, a), l + 1, a);
    for (size_t i = 0; i < r.size(); ++i) r[i] += t[i];
  }
  return r;
}

void spherical_tables(std::vector<double>& tab, std::vector<int>& off) {
  const int LM = 4;
  // S[l][m + l]
  std::vector<std::vector<Poly>> S(LM + 1);
  S[0] = {Poly{1.0}};
  for (int l = 0; l < LM; ++l) {
    S[l + 1].assign(2 * l + 3, Poly(ncart(l + 1), 0.0));
    const double d0 = (l == 0) ? 1.0 : 0.0;
    const double f = std::sqrt(std::pow(2.0, d0) * (2 * l + 1) / (2.0 * l + 2));
    {  // m = l+1 and m = -(l+1)
      Poly xs = mul_axis(S[l][2 * l], l, 0), ys = mul_axis(S[l][2 * l], l, 1);
      Poly& pp = S[l + 1][2 * l + 2];
      Poly& pm = S[l + 1][0];
      for (int i = 0; i < ncart(l + 1); ++i) { pp[i] = f * xs[i]; pm[i] = f * ys[i]; }
      if (l > 0) {
        Poly yn = mul_axis(S[l][0], l, 1), xn = mul_axis(S[l][0], l, 0);
        for (int i = 0; i < ncart(l + 1); ++i) { pp[i] -= f * yn[i]; pm[i] += f * xn[i]; }
      }
    }
    for (int m = -l; m <= l; ++m) {
      Poly zs = mul_axis(S[l][m + l], l, 2);
      Poly& o = S[l + 1][m + l + 1];
      for (int i = 0; i < ncart(l + 1); ++i) o[i] = (2 * l + 1) * zs[i];
      if (l >= 1 && std::abs(m) <= l - 1) {
        Poly r2 = mul_r2(S[l - 1][m + l - 1], l - 1);
        double c = std::sqrt(double((l + m) * (l - m)));
        for (int i = 0; i < ncart(l + 1); ++i) o[i] -= c * r2[i];
      }
      double dn = std::sqrt(double((l + m + 1) * (l - m + 1)));
      for (int i = 0; i < ncart(l + 1); ++i) o[i] /= dn;
    }
  }
  tab.clear();
  off.assign(LM + 2, 0);
  for (int l = 0; l <= LM; ++l) {
    off[l] = (int)tab.size();
    // Cartesian metric of x^l-normalised monomials (same centre/exponent)
    std::vector<int> ex;
    for (int x = l; x >= 0; --x)
      for (int y = l - x; y >= 0; --y) { ex.push_back(x); ex.push_back(y); ex.push_back(l - x - y); }
    const int nc = ncart(l);
    for (int row = 0; row < 2 * l + 1; ++row) {
      int m = (l == 1) ? (row == 0 ? 1 : (row == 1 ? -1 : 0)) : row - l;  // p kept as (x, y, z)
      const Poly& s = S[l][m + l];
      double nrm = 0.0;
      for (int i = 0; i < nc; ++i)
        for (int j = 0; j < nc; ++j) {
          int sx = ex[3 * i] + ex[3 * j], sy = ex[3 * i + 1] + ex[3 * j + 1], sz = ex[3 * i + 2] + ex[3 * j + 2];
          if ((sx | sy | sz) & 1) continue;
          nrm += s[i] * s[j] * dfac(sx - 1) * dfac(sy - 1) * dfac(sz - 1) / dfac(2 * l - 1);
        }
      nrm = 1.0 / std::sqrt(nrm);
      for (int i = 0; i < nc; ++i) tab.push_back(s[i] * nrm);
    }
  }
  off[LM + 1] = (int)tab.size();
}

// ---------------------------------------------------------------------------
// Boys table F_m(k h), composite Gauss-Legendre in long double
// ---------------------------------------------------------------------------
static void gauss_legendre(int n, std::vector<long double>& x, std::vector<long double>& w) {
  x.resize(n);
  w.resize(n);
  const long double pi = 3.141592653589793238462643383279502884L;
  for (int i = 0; i < n; ++i) {
    long double z = cosl(pi * (i + 0.75L) / (n + 0.5L)), dp = 0;
    for (int it = 0; it < 100; ++it) {
      long double p0 = 1, p1 = z;
      for (int k = 2; k <= n; ++k) {
        long double p2 = ((2 * k - 1) * z * p1 - (k - 1) * p0) / k;
        p0 = p1;
        p1 = p2;
      }
      dp = n * (z * p1 - p0) / (z * z - 1);
      long double dz = p1 / dp;
      z -= dz;
      if (fabsl(dz) < 1e-19L) break;
    }
    x[i] = z;
    w[i] = 2 / ((1 - z * z) * dp * dp);
  }
}

void boys_table(std::vector<double>& tab) {
  const int NP = 64, NG = 14;
  std::vector<long double> gx, gw;
  gauss_legendre(NG, gx, gw);
  tab.assign(BOYS_TABLE_DOUBLES, 0.0);
  std::vector<long double> acc(BOYS_NM);
  for (int k = 0; k < BOYS_NGRID; ++k) {
    long double T = (long double)k * (long double)BOYS_H;
    std::fill(acc.begin(), acc.end(), 0.0L);
    for (int pnl = 0; pnl < NP; ++pnl) {
      long double a = (long double)pnl / NP, b = (long double)(pnl + 1) / NP;
      for (int i = 0; i < NG; ++i) {
        long double t = 0.5L * (b - a) * gx[i] + 0.5L * (a + b);
        long double wt = 0.5L * (b - a) * gw[i] * expl(-T * t * t);
        long double t2 = t * t, pw = 1.0L;
        for (int m = 0; m < BOYS_NM; ++m) {
          acc[m] += wt * pw;
          pw *= t2;
        }
      }
    }
    for (int L = 0; L < BOYS_LTAB; ++L) {
      double* row = tab.data() + ((size_t)L * BOYS_NGRID + k) * BOYS_ROW;
      for (int j = 0; j < BOYS_TAYLOR; ++j) row[j] = (double)acc[L + j];
      row[BOYS_ROW - 1] = (double)expl(-T);
    }
  }
  for (int k = 0; k < BOYS_NEXP; ++k)
    tab[BOYS_EXP_OFF + k] = (double)expl(-(40.0L + (long double)k * (long double)BOYS_H));
}

}  // namespace mako

using namespace mako;

static bool is_fin(double v) { return std::isfinite(v); }

template <class T>
static mako_status upload(DevBuf& d, const std::vector<T>& h) {
  mako_status st = d.alloc(h.size() * sizeof(T));
  if (st) return st;
  if (!h.empty()) {
    cudaError_t e = cudaMemcpy(d.p, h.data(), h.size() * sizeof(T), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) return fail(MAKO_ERR_CUDA, std::string("cudaMemcpy: ") + cudaGetErrorString(e));
  }
  return MAKO_OK;
}

extern "C" mako_status mako_basis_create(int natm, const int* Z, const double* xyz, int nshell, const int* shell_atom,
                                         const int* shell_l, const int* shell_nprim, const double* exps,
                                         const double* coefs, int pure, mako_basis* out) {
  try {
    if (!out) return fail(MAKO_ERR_INVALID, "out is NULL");
    *out = nullptr;
    if (natm < 1 || nshell < 1 || !Z || !xyz || !shell_atom || !shell_l || !shell_nprim || !exps || !coefs)
      return fail(MAKO_ERR_INVALID, "NULL pointer or empty molecule/basis");
    if (pure != 1) return fail(MAKO_ERR_UNSUPPORTED, "only pure (spherical) functions are supported (pure=1)");
    for (int i = 0; i < 3 * natm; ++i)
      if (!is_fin(xyz[i])) return fail(MAKO_ERR_INVALID, "non-finite atom coordinate");
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
      return fail(MAKO_ERR_CUDA, "no CUDA device (there is no CPU fallback)");
    std::unique_ptr<mako_basis_s> B(new mako_basis_s);
    cudaGetDevice(&B->device);
    B->natm = natm;
    B->Z.assign(Z, Z + natm);
    B->axyz.assign(xyz, xyz + 3 * natm);
    B->nshell = nshell;
    B->pure = 1;
    int np = 0, nb = 0;
    for (int s = 0; s < nshell; ++s) {
      if (shell_atom[s] < 0 || shell_atom[s] >= natm) return fail(MAKO_ERR_INVALID, "shell_atom out of range");
      if (shell_l[s] < 0) return fail(MAKO_ERR_INVALID, "negative l");
      if (shell_l[s] > LMAX) return fail(MAKO_ERR_UNSUPPORTED, "l > MAKO_LMAX");
      if (shell_nprim[s] < 1) return fail(MAKO_ERR_INVALID, "nprim < 1");
      B->atom.push_back(shell_atom[s]);
      B->l.push_back(shell_l[s]);
      B->nprim.push_back(shell_nprim[s]);
      B->poff.push_back(np);
      B->ao.push_back(nb);
      for (int k = 0; k < 3; ++k) B->sxyz.push_back(xyz[3 * shell_atom[s] + k]);
      np += shell_nprim[s];
      nb += nsph(shell_l[s]);
    }
    B->poff.push_back(np);
    B->ao.push_back(nb);
    B->nbf = nb;
    for (int i = 0; i < np; ++i)
      if (!is_fin(exps[i]) || !(exps[i] > 0) || !is_fin(coefs[i]))
        return fail(MAKO_ERR_INVALID, "exponents must be finite and > 0; coefficients finite");
    B->exps.assign(exps, exps + np);
    B->cn.resize(np);
    const double pi = 3.14159265358979323846;
    for (int s = 0; s < nshell; ++s) {
      const int l = B->l[s], o = B->poff[s], k = B->nprim[s];
      // primitive norm of the x^l component: <x^l e^{-a r^2}|x^l e^{-a r^2}> = (2l-1)!!/(4a)^l (pi/2a)^{3/2}
      for (int i = 0; i < k; ++i) {
        double a = exps[o + i];
        double n2 = dfac(2 * l - 1) / std::pow(4.0 * a, l) * std::pow(pi / (2.0 * a), 1.5);
        B->cn[o + i] = coefs[o + i] / std::sqrt(n2);
      }
      double S = 0.0;
      for (int i = 0; i < k; ++i)
        for (int j = 0; j < k; ++j) {
          double p = exps[o + i] + exps[o + j];
          S += B->cn[o + i] * B->cn[o + j] * dfac(2 * l - 1) / std::pow(2.0 * p, l) * std::pow(pi / p, 1.5);
        }
      if (!(S > 0) || !is_fin(S)) return fail(MAKO_ERR_INVALID, "contracted shell has zero norm");
      for (int i = 0; i < k; ++i) B->cn[o + i] /= std::sqrt(S);
    }
    std::vector<double> sph, boys;
    spherical_tables(sph, B->sph_off);
    boys_table(boys);
    std::vector<int> aos(B->ao.begin(), B->ao.end() - 1);
    mako_status st;
    if ((st = upload(B->d_ao, aos)) || (st = upload(B->d_sxyz, B->sxyz)) || (st = upload(B->d_l, B->l)) ||
        (st = upload(B->d_poff, B->poff)) || (st = upload(B->d_exps, B->exps)) || (st = upload(B->d_cn, B->cn)) ||
        (st = upload(B->d_sph, sph)) || (st = upload(B->d_boys, boys)))
      return st;
    // pageable cudaMemcpy may return before its DMA lands; the pair builder runs on the caller's
    // (possibly non-blocking) stream: finish the uploads here
    if (cudaDeviceSynchronize() != cudaSuccess) return fail(MAKO_ERR_CUDA, "basis upload");
    *out = B.release();
    return MAKO_OK;
  } catch (const std::exception& e) {
    return fail(MAKO_ERR_OOM, std::string("host exception: ") + e.what());
  }
}

extern "C" mako_status mako_basis_nbf(mako_basis b, int* nbf) {
  if (!b || !nbf) return fail(MAKO_ERR_INVALID, "NULL argument");
  *nbf = b->nbf;
  return MAKO_OK;
}
extern "C" mako_status mako_basis_nshell(mako_basis b, int* n) {
  if (!b || !n) return fail(MAKO_ERR_INVALID, "NULL argument");
  *n = b->nshell;
  return MAKO_OK;
}
extern "C" mako_status mako_basis_ao_offsets(mako_basis b, int* ao) {
  if (!b || !ao) return fail(MAKO_ERR_INVALID, "NULL argument");
  std::memcpy(ao, b->ao.data(), sizeof(int) * (b->nshell + 1));
  return MAKO_OK;
}
extern "C" void mako_basis_destroy(mako_basis b) { delete b; }

extern "C" const char* mako_last_error(void) { return mako::last_error_cstr(); }
extern "C" const char* mako_version(void) { return "mako-b200 0.1 (sm_100a, FP64 DMMA)"; }
