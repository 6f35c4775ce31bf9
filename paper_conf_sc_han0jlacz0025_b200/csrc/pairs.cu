// pairs.cu -- shell-pair data: Hermite expansion matrices E~_ab on the device,
// Schwarz factors from the diagonal ERIs, screening, bucketing by (la, lb), Q-sorted order.
//
// E~_ab (the "E_AB" input of PAPER.md Alg. 1) for primitive pair (alpha at A, beta at B):
//   p = alpha + beta, P = (alpha A + beta B)/p, mu = alpha beta / p
//   1D McMurchie-Davidson recursion per axis (Helgaker et al. Eq. 9.5.6):
//     E^{00}_0 = exp(-mu X_AB^2)
//     E^{i+1,j}_t = E^{ij}_{t-1}/(2p) + X_PA E^{ij}_t + (t+1) E^{ij}_{t+1}
//     E^{i,j+1}_t = E^{ij}_{t-1}/(2p) + X_PB E^{ij}_t + (t+1) E^{ij}_{t+1}
//   E~[(sa sb)][(tuv)] = (c_i c_j / p) sum_{ca,cb} C_a[sa][ca] C_b[sb][cb] E^x_t E^y_u E^z_v
// so that (ab|cd) = sum_{ij,kl} sum_{p,q} E~_ab[p] (-1)^{|q|} R_{p+q} E~_cd[q] with the
// 2 pi^{5/2}/sqrt(p+q) factor carried by the R seed (eri_core.cuh).
#include <algorithm>
#include <cmath>
#include <numeric>

#include "eri_kernels.cuh"

namespace mako {

__device__ __forceinline__ void cart_decode(int l, int c, int& x, int& y, int& z) {
  // inverse of cart_index: c = (y+z)(y+z+1)/2 + z
  int s = 0;
  while ((s + 1) * (s + 2) / 2 <= c) ++s;
  z = c - s * (s + 1) / 2;
  y = s - z;
  x = l - s;
}

__device__ __forceinline__ void herm_decode(int e, int& t, int& u, int& v) {
  int k = 0;
  while (nH(k) <= e) ++k;
  int r = e - nH(k - 1);
  int s = 0;
  while ((s + 1) * (s + 2) / 2 <= r) ++s;
  v = r - s * (s + 1) / 2;
  u = s - v;
  t = k - s;
}

// one CTA per primitive pair
__global__ void build_E_kernel(int la, int lb, int nprim, const int* __restrict__ pshA, const int* __restrict__ pshB,
                               const int* __restrict__ pi, const int* __restrict__ pj,
                               const double* __restrict__ sxyz, const double* __restrict__ exps,
                               const double* __restrict__ cn, const int* __restrict__ spoff,
                               const double* __restrict__ sph, int sphA, int sphB, double* __restrict__ pdat,
                               double* __restrict__ Ebra, double* __restrict__ Eket) {
  const int id = blockIdx.x;
  if (id >= nprim) return;
  __shared__ double E1[3][LMAX + 1][LMAX + 1][2 * LMAX + 1];
  __shared__ double pref_s;
  const int sA = pshA[id], sB = pshB[id];
  const int ia = spoff[sA] + pi[id], ib = spoff[sB] + pj[id];
  const double al = exps[ia], be = exps[ib], p = al + be;
  for (int o = threadIdx.x; o < 3 * (LMAX + 1) * (LMAX + 1) * (2 * LMAX + 1); o += blockDim.x)
    (&E1[0][0][0][0])[o] = 0.0;
  __syncthreads();
  if (threadIdx.x < 3) {
    const int d = threadIdx.x;
    const double A = sxyz[3 * sA + d], B = sxyz[3 * sB + d];
    const double P = (al * A + be * B) / p, XPA = P - A, XPB = P - B, XAB = A - B;
    const double h = 0.5 / p;
    E1[d][0][0][0] = exp(-al * be / p * XAB * XAB);
    for (int i = 0; i <= la; ++i)
      for (int j = 0; j <= lb; ++j) {
        if (i == 0 && j == 0) continue;
        const bool up_i = (j == 0);
        const int i0 = up_i ? i - 1 : i, j0 = up_i ? j : j - 1;
        const double X = up_i ? XPA : XPB;
        for (int t = 0; t <= i + j; ++t) {
          double v = X * E1[d][i0][j0][t];
          if (t > 0) v += h * E1[d][i0][j0][t - 1];
          if (t + 1 <= i0 + j0) v += (t + 1) * E1[d][i0][j0][t + 1];
          E1[d][i][j][t] = v;
        }
      }
    if (d == 0) {
      pref_s = cn[ia] * cn[ib] / p;
      pdat[4 * id] = p;
    }
    pdat[4 * id + 1 + d] = P;
  }
  __syncthreads();
  const int nsa = 2 * la + 1, nsb = 2 * lb + 1, nab = nsa * nsb, nh = nH(la + lb);
  const int nca = ncart(la), ncb = ncart(lb);
  const double pref = pref_s;
  for (int o = threadIdx.x; o < nab * nh; o += blockDim.x) {
    const int ab = o / nh, h = o % nh, sa = ab / nsb, sb = ab % nsb;
    int t, u, v;
    herm_decode(h, t, u, v);
    double s = 0.0;
    for (int ca = 0; ca < nca; ++ca) {
      const double cA = sph[sphA + sa * nca + ca];
      if (cA == 0.0) continue;
      int ax, ay, az;
      cart_decode(la, ca, ax, ay, az);
      for (int cb = 0; cb < ncb; ++cb) {
        const double cB = sph[sphB + sb * ncb + cb];
        if (cB == 0.0) continue;
        int bx, by, bz;
        cart_decode(lb, cb, bx, by, bz);
        if (t > ax + bx || u > ay + by || v > az + bz) continue;
        s += cA * cB * E1[0][ax][bx][t] * E1[1][ay][by][u] * E1[2][az][bz][v];
      }
    }
    const double val = s * pref;
    Ebra[(size_t)id * nab * nh + (size_t)ab * nh + h] = val;
    Eket[(size_t)id * nab * nh + (size_t)h * nab + ab] = ((t + u + v) & 1) ? -val : val;
  }
}

static mako_status cuda_check(cudaError_t e, const char* what) {
  if (e != cudaSuccess) return fail(MAKO_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
  return MAKO_OK;
}

template <class T>
static mako_status upload_async(DevBuf& d, const std::vector<T>& h, cudaStream_t s) {
  mako_status st = d.alloc(h.size() * sizeof(T));
  if (st) return st;
  if (!h.empty()) return cuda_check(cudaMemcpyAsync(d.p, h.data(), h.size() * sizeof(T), cudaMemcpyHostToDevice, s),
                                    "cudaMemcpyAsync");
  return MAKO_OK;
}

PairView PairBucket::view() const {
  PairView v;
  v.n = n();
  v.la = la;
  v.lb = lb;
  v.shA = d_shA.as<int>();
  v.shB = d_shB.as<int>();
  v.Q = d_Q.as<double>();
  v.poff = d_poff.as<int>();
  v.pdat = d_pdat.as<double>();
  v.Ebra = d_Ebra.as<double>();
  v.Eket = d_Eket.as<double>();
  v.EbraD = d_EbraD.as<double>();
  v.EketD = d_EketD.as<double>();
  v.EbraF = d_EbraF.as<float>();
  v.EketF = d_EketF.as<float>();
  return v;
}

// FP64 copies of E~ in mma.m8n8k4 fragment order, zero-padded: A fragments of GEMM1 (lane (g,t):
// E~[8m+g][4k+t]) and B fragment pairs of GEMM2 (lane (g,t): Ek[8n+2t][8j+g], Ek[8n+2t+1][8j+g]).
// One thread per output double.
__global__ void build_frag_kernel(int nab, int nh, long long total_a, long long total_b, const double* __restrict__ Ebra,
                                  const double* __restrict__ Eket, double* __restrict__ EbraD,
                                  double* __restrict__ EketD) {
  const int MT = (nab + 7) / 8, KS = (nh + 3) / 4, NQ = (nh + 7) / 8, NC = (nab + 7) / 8;
  const int AF = MT * KS * 32, BF = NQ * NC * 64;
  for (long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x; x < total_a + total_b;
       x += (long long)gridDim.x * blockDim.x) {
    double v = 0.0;
    if (x < total_a) {
      const long long id = x / AF;
      const int r = (int)(x % AF), mk = r / 32, lane = r % 32;
      const int m = mk / KS, k = mk % KS, g = lane >> 2, t = lane & 3;
      const int row = 8 * m + g, col = 4 * k + t;
      if (row < nab && col < nh) v = Ebra[(size_t)id * nab * nh + (size_t)row * nh + col];
      EbraD[x] = v;
    } else {
      const long long y = x - total_a, id = y / BF;
      const int r = (int)(y % BF), nj = r / 64, lane = (r % 64) / 2, e = r % 2;
      const int n = nj / NC, j = nj % NC, g = lane >> 2, t = lane & 3;
      const int q = 8 * n + 2 * t + e, cd = 8 * j + g;
      if (q < nh && cd < nab) v = Eket[(size_t)id * nab * nh + (size_t)q * nab + cd];
      EketD[y] = v;
    }
  }
}

// Build device pair data for the given per-bucket shell lists (A has the higher l).
// Primitive pairs with exp(-mu |AB|^2) < PRIM_PAIR_EPS are dropped (reading R7); a
// shell pair keeps at least... nothing: pairs with zero surviving primitive pairs get an empty range.
mako_status build_pair_set(const mako_basis_s* B, const std::vector<int> (&A)[NBUCKET],
                           const std::vector<int> (&Bs)[NBUCKET], PairSet& out, void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  for (int b = 0; b < NBUCKET; ++b) {
    PairBucket& pb = out.b[b];
    pb.la = bucket_la(b);
    pb.lb = bucket_lb(b);
    pb.shA = A[b];
    pb.shB = Bs[b];
    pb.Q.assign(pb.shA.size(), 0.0);
    pb.poff.assign(1, 0);
    std::vector<int> psA, psB, ppi, ppj;
    for (size_t k = 0; k < pb.shA.size(); ++k) {
      const int sA = pb.shA[k], sB = pb.shB[k];
      double R2 = 0;
      for (int d = 0; d < 3; ++d) {
        double x = B->sxyz[3 * sA + d] - B->sxyz[3 * sB + d];
        R2 += x * x;
      }
      for (int i = 0; i < B->nprim[sA]; ++i)
        for (int j = 0; j < B->nprim[sB]; ++j) {
          const double a = B->exps[B->poff[sA] + i], c = B->exps[B->poff[sB] + j];
          if (std::exp(-a * c / (a + c) * R2) < PRIM_PAIR_EPS) continue;
          psA.push_back(sA); psB.push_back(sB); ppi.push_back(i); ppj.push_back(j);
        }
      pb.poff.push_back((int)psA.size());
    }
    const int np = (int)psA.size();
    const size_t esz = (size_t)nsph(pb.la) * nsph(pb.lb) * nH(pb.la + pb.lb);
    mako_status st;
    DevBuf dA, dB, di, dj;
    if ((st = upload_async(pb.d_shA, pb.shA, s)) || (st = upload_async(pb.d_shB, pb.shB, s)) ||
        (st = upload_async(pb.d_Q, pb.Q, s)) || (st = upload_async(pb.d_poff, pb.poff, s)) ||
        (st = pb.d_pdat.alloc(sizeof(double) * 4 * (size_t)std::max(np, 1))) ||
        (st = pb.d_Ebra.alloc(sizeof(double) * esz * std::max(np, 1))) ||
        (st = pb.d_Eket.alloc(sizeof(double) * esz * std::max(np, 1))) || (st = upload_async(dA, psA, s)) ||
        (st = upload_async(dB, psB, s)) || (st = upload_async(di, ppi, s)) || (st = upload_async(dj, ppj, s)))
      return st;
    if (np > 0) {
      build_E_kernel<<<np, 128, 0, s>>>(pb.la, pb.lb, np, dA.as<int>(), dB.as<int>(), di.as<int>(), dj.as<int>(),
                                        B->d_sxyz.as<double>(), B->d_exps.as<double>(), B->d_cn.as<double>(),
                                        B->d_poff.as<int>(), B->d_sph.as<double>(), B->sph_off[pb.la],
                                        B->sph_off[pb.lb], pb.d_pdat.as<double>(), pb.d_Ebra.as<double>(),
                                        pb.d_Eket.as<double>());
      if ((st = cuda_check(cudaGetLastError(), "build_E_kernel"))) return st;
    }
    {
      const long long ta = (long long)std::max(np, 1) * frag_a_doubles(pb.la, pb.lb);
      const long long tb = (long long)std::max(np, 1) * frag_b_doubles(pb.la, pb.lb);
      if ((st = pb.d_EbraD.alloc(sizeof(double) * ta)) || (st = pb.d_EketD.alloc(sizeof(double) * tb))) return st;
      if (np > 0) {
        build_frag_kernel<<<1184, 256, 0, s>>>(nsph(pb.la) * nsph(pb.lb), nH(pb.la + pb.lb), ta, tb,
                                               pb.d_Ebra.as<double>(), pb.d_Eket.as<double>(), pb.d_EbraD.as<double>(),
                                               pb.d_EketD.as<double>());
        if ((st = cuda_check(cudaGetLastError(), "build_frag_kernel"))) return st;
      }
    }
    // temporaries are freed at scope exit: make sure the kernel is done with them
    if ((st = cuda_check(cudaStreamSynchronize(s), "build_pair_set sync"))) return st;
  }
  return MAKO_OK;
}

// TF32 copies of E~ in mma.m16n8k8 fragment order (reduced-precision tier, eri_quant.cuh), zero
// padded: A fragments of GEMM1 (lane (g,t): E~[16m+g][8k+t], E~[16m+g+8][8k+t], E~[16m+g][8k+t+4],
// E~[16m+g+8][8k+t+4]) and B fragments of GEMM2 (lane (g,t): Ek[8n+2t][8j+g], Ek[8n+2t+1][8j+g],
// Ek = (-1)^{|q|} E~^T).  One thread per output float.
__global__ void build_lowp_kernel(int nab, int nh, long long total_a, long long total_b, const double* __restrict__ Ebra,
                                  const double* __restrict__ Eket, float* __restrict__ EbraF,
                                  float* __restrict__ EketF) {
  const int MT = (nab + 15) / 16, KS = (nh + 7) / 8, NQ = (nh + 7) / 8, NC = (nab + 7) / 8;
  const int AF = MT * KS * 128, BF = NQ * NC * 64;
  for (long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x; x < total_a + total_b;
       x += (long long)gridDim.x * blockDim.x) {
    double v = 0.0;
    if (x < total_a) {
      const long long id = x / AF;
      const int r = (int)(x % AF), mk = r / 128, lane = (r % 128) / 4, e = r % 4;
      const int m = mk / KS, k = mk % KS, g = lane >> 2, t = lane & 3;
      const int row = 16 * m + g + ((e & 1) ? 8 : 0), col = 8 * k + t + ((e & 2) ? 4 : 0);
      if (row < nab && col < nh) v = Ebra[(size_t)id * nab * nh + (size_t)row * nh + col];
      unsigned u;
      asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(u) : "f"((float)v));
      EbraF[x] = __uint_as_float(u);
    } else {
      const long long y = x - total_a, id = y / BF;
      const int r = (int)(y % BF), nj = r / 64, lane = (r % 64) / 2, e = r % 2;
      const int n = nj / NC, j = nj % NC, g = lane >> 2, t = lane & 3;
      const int q = 8 * n + 2 * t + e, cd = 8 * j + g;
      if (q < nh && cd < nab) v = Eket[(size_t)id * nab * nh + (size_t)q * nab + cd];
      unsigned u;
      asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(u) : "f"((float)v));
      EketF[y] = __uint_as_float(u);
    }
  }
}

mako_status ensure_lowp(PairSet& set, void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  for (int b = 0; b < NBUCKET; ++b) {
    PairBucket& pb = set.b[b];
    if (pb.d_EbraF.p) continue;
    // an empty bucket keeps a one-element allocation and no kernel (its E~ was never written)
    const long long np = std::max(pb.poff.empty() ? 0 : pb.poff.back(), 1);
    const bool empty = pb.poff.empty() || pb.poff.back() == 0;
    const int nab = nsph(pb.la) * nsph(pb.lb), nh = nH(pb.la + pb.lb);
    const long long ta = np * lowp_a_floats(pb.la, pb.lb), tb = np * lowp_b_floats(pb.la, pb.lb);
    mako_status st;
    if ((st = pb.d_EbraF.alloc(sizeof(float) * ta)) || (st = pb.d_EketF.alloc(sizeof(float) * tb))) return st;
    if (empty) continue;
    build_lowp_kernel<<<1184, 256, 0, s>>>(nab, nh, ta, tb, pb.d_Ebra.as<double>(), pb.d_Eket.as<double>(),
                                          pb.d_EbraF.as<float>(), pb.d_EketF.as<float>());
    if ((st = cuda_check(cudaGetLastError(), "build_lowp_kernel"))) return st;
  }
  return MAKO_OK;
}

// Q_ab = sqrt(max |(ab|ab)|) for every pair of the set (diagonal quartets through the class kernels)
mako_status compute_schwarz(const mako_basis_s* B, PairSet& set, void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  for (int b = 0; b < NBUCKET; ++b) {
    PairBucket& pb = set.b[b];
    const int n = pb.n();
    if (n == 0) continue;
    std::vector<int> idx(n);
    std::iota(idx.begin(), idx.end(), 0);
    std::vector<long long> qo(idx.begin(), idx.end());
    DevBuf di, dq;
    mako_status st;
    if ((st = upload_async(di, idx, s)) || (st = upload_async(dq, qo, s))) return st;
    BatchArgs a{};
    a.bra = a.ket = pb.view();
    a.nq = n;
    a.qbra = a.qket = di.as<int>();
    a.qout = dq.as<long long>();
    a.qflag = nullptr;
    a.out = pb.d_Q.as<double>();
    a.boys = B->d_boys.as<double>();
    a.diag = 1;
    if ((st = launch_batch_class(b, b, a, stream))) return st;
    if ((st = cuda_check(cudaMemcpyAsync(pb.Q.data(), pb.d_Q.p, sizeof(double) * n, cudaMemcpyDeviceToHost, s),
                         "Q download")))
      return st;
    if ((st = cuda_check(cudaStreamSynchronize(s), "schwarz sync"))) return st;
  }
  return MAKO_OK;
}

}  // namespace mako

using namespace mako;

extern "C" mako_status mako_shellpairs_screen(mako_basis basis, double thresh, void* cuda_stream, mako_pairs* out) {
  try {
    if (!basis || !out) return fail(MAKO_ERR_INVALID, "NULL argument");
    *out = nullptr;
    if (!(thresh >= 0) || !std::isfinite(thresh)) return fail(MAKO_ERR_INVALID, "thresh must be finite and >= 0");
    int dev = -1;
    cudaGetDevice(&dev);
    if (dev != basis->device) return fail(MAKO_ERR_STATE, "basis belongs to another CUDA device");
    // 1. candidate pairs: (A, B) with l_A > l_B, or l_A == l_B and A >= B
    std::vector<int> A[NBUCKET], Bs[NBUCKET];
    for (int a = 0; a < basis->nshell; ++a)
      for (int b = 0; b < basis->nshell; ++b) {
        const int la = basis->l[a], lb = basis->l[b];
        if (la < lb || (la == lb && a < b)) continue;
        A[bucket_of(la, lb)].push_back(a);
        Bs[bucket_of(la, lb)].push_back(b);
      }
    PairSet cand;
    mako_status st;
    if ((st = build_pair_set(basis, A, Bs, cand, cuda_stream))) return st;
    if ((st = compute_schwarz(basis, cand, cuda_stream))) return st;
    // 2. screening Q_ab * Q_max >= thresh, pairs without primitive pairs dropped; sort by Q desc
    double qmax = 0;
    for (int b = 0; b < NBUCKET; ++b)
      for (double q : cand.b[b].Q) qmax = std::max(qmax, q);
    std::unique_ptr<mako_pairs_s> P(new mako_pairs_s);
    P->basis = basis;
    P->tau = thresh;
    std::vector<int> A2[NBUCKET], B2[NBUCKET];
    std::vector<double> Q2[NBUCKET];
    std::vector<int> seg[NBUCKET];
    for (int b = 0; b < NBUCKET; ++b) {
      const PairBucket& cb = cand.b[b];
      std::vector<int> keep;
      for (int k = 0; k < cb.n(); ++k)
        if (cb.poff[k + 1] > cb.poff[k] && cb.Q[k] > 0 && cb.Q[k] * qmax >= thresh) keep.push_back(k);
      auto grp = [&](int k) { return kgroup(cb.poff[k + 1] - cb.poff[k]); };
      std::stable_sort(keep.begin(), keep.end(), [&](int x, int y) {
        const int gx = grp(x), gy = grp(y);
        return gx != gy ? gx < gy : cb.Q[x] > cb.Q[y];
      });
      seg[b].assign(NKGROUP + 1, 0);
      for (int k : keep) {
        A2[b].push_back(cb.shA[k]);
        B2[b].push_back(cb.shB[k]);
        Q2[b].push_back(cb.Q[k]);
        seg[b][grp(k) + 1]++;
      }
      for (int g = 0; g < NKGROUP; ++g) seg[b][g + 1] += seg[b][g];
    }
    for (int b = 0; b < NBUCKET; ++b) {  // free candidate device memory before the rebuild
      cand.b[b].d_Ebra.release();
      cand.b[b].d_Eket.release();
      cand.b[b].d_EbraD.release();
      cand.b[b].d_EketD.release();
    }
    if ((st = build_pair_set(basis, A2, B2, P->set, cuda_stream))) return st;
    cudaStream_t s = (cudaStream_t)cuda_stream;
    for (int b = 0; b < NBUCKET; ++b) {
      P->set.b[b].Q = Q2[b];
      P->set.b[b].seg = seg[b];
      if ((st = upload_async(P->set.b[b].d_Q, Q2[b], s))) return st;
    }
    if ((st = P->d_counters.alloc(sizeof(unsigned long long) * 2 * NCLASS))) return st;
    if ((st = cuda_check(cudaStreamSynchronize(s), "screen sync"))) return st;
    *out = P.release();
    return MAKO_OK;
  } catch (const std::exception& e) {
    return fail(MAKO_ERR_OOM, std::string("host exception: ") + e.what());
  }
}

extern "C" void mako_pairs_destroy(mako_pairs p) { delete p; }
