// jk.cu -- mako_build_jk (the hot path), per-threshold quartet plans, sharding, eri_batch, boys.
//
// Plan: classes (X|Y) over pair buckets X >= Y (55 for l <= 3, 120 for l <= 4).  Within a
// bucket pairs are sorted by Q descending, so for bra P the kets with Q_P Q_R >= thresh are a
// PREFIX of bucket Y (clipped to R <= P when X == Y: canonical ab >= cd).  A task is (P, <= KT
// consecutive kets of that prefix); tasks of a class are numbered by a prefix sum over P.
// Sharding: shard s of n takes tasks [T s/n, T (s+1)/n) of every class.
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <limits>

#include "eri_kernels.cuh"
#include "eri_core.cuh"
#include "eri_kf.cuh"
#include "eri_slab.cuh"

namespace mako {

// ----- dispatch over the 55 classes ----------------------------------------
#define MAKO_CLASS_LIST(F)                                                                                        \
  F(0, 0) F(1, 0) F(1, 1) F(2, 0) F(2, 1) F(2, 2) F(3, 0) F(3, 1) F(3, 2) F(3, 3) F(4, 0) F(4, 1) F(4, 2)          \
  F(4, 3) F(4, 4) F(5, 0) F(5, 1) F(5, 2) F(5, 3) F(5, 4) F(5, 5) F(6, 0) F(6, 1) F(6, 2) F(6, 3) F(6, 4)          \
  F(6, 5) F(6, 6) F(7, 0) F(7, 1) F(7, 2) F(7, 3) F(7, 4) F(7, 5) F(7, 6) F(7, 7) F(8, 0) F(8, 1) F(8, 2)          \
  F(8, 3) F(8, 4) F(8, 5) F(8, 6) F(8, 7) F(8, 8) F(9, 0) F(9, 1) F(9, 2) F(9, 3) F(9, 4) F(9, 5) F(9, 6)          \
  F(9, 7) F(9, 8) F(9, 9) F(10, 0) F(10, 1) F(10, 2) F(10, 3) F(10, 4) F(10, 5) F(10, 6) F(10, 7) F(10, 8)         \
  F(10, 9) F(10, 10) F(11, 0) F(11, 1) F(11, 2) F(11, 3) F(11, 4) F(11, 5) F(11, 6) F(11, 7) F(11, 8) F(11, 9)     \
  F(11, 10) F(11, 11) F(12, 0) F(12, 1) F(12, 2) F(12, 3) F(12, 4) F(12, 5) F(12, 6) F(12, 7) F(12, 8) F(12, 9)    \
  F(12, 10) F(12, 11) F(12, 12) F(13, 0) F(13, 1) F(13, 2) F(13, 3) F(13, 4) F(13, 5) F(13, 6) F(13, 7) F(13, 8)   \
  F(13, 9) F(13, 10) F(13, 11) F(13, 12) F(13, 13) F(14, 0) F(14, 1) F(14, 2) F(14, 3) F(14, 4) F(14, 5)           \
  F(14, 6) F(14, 7) F(14, 8) F(14, 9) F(14, 10) F(14, 11) F(14, 12) F(14, 13) F(14, 14)

mako_status launch_jk_class(int X, int Y, const JKArgs& a, void* stream, int* nl) {
#define MAKO_JK_CASE(x, y) \
  if (X == x && Y == y) return launch_jk_xy<x, y>(a, stream, nl);
  MAKO_CLASS_LIST(MAKO_JK_CASE)
#undef MAKO_JK_CASE
  return fail(MAKO_ERR_UNSUPPORTED, "unknown class");
}

mako_status launch_batch_class(int X, int Y, const BatchArgs& a, void* stream) {
#define MAKO_B_CASE(x, y) \
  if (X == x && Y == y) return launch_batch_xy<x, y>(a, stream);
  MAKO_CLASS_LIST(MAKO_B_CASE)
#undef MAKO_B_CASE
  return fail(MAKO_ERR_UNSUPPORTED, "unknown class");
}

static int class_task_kets(int X, int Y) {
#define MAKO_KT_CASE(x, y) \
  if (X == x && Y == y) return task_kets_xy<x, y>();
  MAKO_CLASS_LIST(MAKO_KT_CASE)
#undef MAKO_KT_CASE
  return 16;
}

static bool class_swap(int X, int Y) {
#define MAKO_SW_CASE(x, y) \
  if (X == x && Y == y) return swap_xy<x, y>();
  MAKO_CLASS_LIST(MAKO_SW_CASE)
#undef MAKO_SW_CASE
  return false;
}

// kernel family of a class (include/mako.h mako_class_family): 0 lane-per-ket (tpq), 1 ket-first (kf),
// 2 ket-first transposed, 3 slot-batched (slab), 4 warp-per-quartet (jk), 5 warp-per-quartet transposed
template <int X, int Y>
static int family_xy() {
  if constexpr (use_kf_swap<X, Y>()) return 2;
  else if constexpr (use_jk_swap<X, Y>()) return 5;
  else if constexpr (use_kf<X, Y>()) return 1;
  else if constexpr (use_tpq(X, Y)) return 0;
  else if constexpr (use_slab<X, Y>()) return 3;
  else return 4;
}
static int class_family(int X, int Y) {
#define MAKO_FAM_CASE(x, y) \
  if (X == x && Y == y) return family_xy<x, y>();
  MAKO_CLASS_LIST(MAKO_FAM_CASE)
#undef MAKO_FAM_CASE
  return -1;
}

bool class_has_lowp(int X, int Y) {
#define MAKO_LP_CASE(x, y) \
  if (X == x && Y == y) return lowp_xy<x, y>();
  MAKO_CLASS_LIST(MAKO_LP_CASE)
#undef MAKO_LP_CASE
  return false;
}

static mako_status cuda_check(cudaError_t e, const char* what) {
  if (e != cudaSuccess) return fail(MAKO_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
  return MAKO_OK;
}

template <class T>
static mako_status upload(DevBuf& d, const std::vector<T>& h) {
  mako_status st = d.alloc(h.size() * sizeof(T));
  if (st) return st;
  if (!h.empty()) return cuda_check(cudaMemcpy(d.p, h.data(), h.size() * sizeof(T), cudaMemcpyHostToDevice), "upload");
  return MAKO_OK;
}

// stream-ordered upload (the kernels reading the buffer are launched on the same stream afterwards;
// a pageable source is staged before cudaMemcpyAsync returns, so `h` may die right after)
template <class T>
static mako_status upload_async(DevBuf& d, const std::vector<T>& h, cudaStream_t s) {
  mako_status st = d.alloc(h.size() * sizeof(T));
  if (st) return st;
  if (!h.empty())
    return cuda_check(cudaMemcpyAsync(d.p, h.data(), h.size() * sizeof(T), cudaMemcpyHostToDevice, s), "upload");
  return MAKO_OK;
}

// number of kets R in [lo, hi) of bucket Y (Q-sorted desc within the segment) with QP * Q[R] >= thresh
static int prefix_count(const std::vector<double>& QY, int lo0, int hi0, double QP, double thresh) {
  int lo = lo0, hi = hi0;
  while (lo < hi) {
    int mid = (lo + hi) / 2;
    if (QP * QY[mid] >= thresh) lo = mid + 1; else hi = mid;
  }
  return lo - lo0;
}

// entries of class plan c for the kets with lo <= Q_P Q_R < hi (hi = +inf: the plain Schwarz prefix);
// in a Q-sorted segment that is the range [prefix(hi), prefix(lo)) of the segment
static mako_status build_class_plan(ClassPlan& c, const PairBucket& bx, const PairBucket& by, bool same, double lo,
                                    double hi) {
  const int nbra = bx.n(), G = NKGROUP;
  c.ent_P.clear();
  c.kbeg.clear();
  c.kend.clear();
  c.task_off.assign(1, 0);
  c.nquartet = 0;
  for (int p = 0; p < nbra; ++p)
    for (int g = 0; g < G; ++g) {
      const int s0 = by.seg.empty() ? 0 : by.seg[g], s1 = by.seg.empty() ? (g == 0 ? by.n() : 0) : by.seg[g + 1];
      if (s1 <= s0) continue;
      int nk = prefix_count(by.Q, s0, s1, bx.Q[p], lo);
      int nh = std::isinf(hi) ? 0 : prefix_count(by.Q, s0, s1, bx.Q[p], hi);
      if (same) {  // canonical: ket position <= bra position
        nk = std::min(nk, std::max(0, p - s0 + 1));
        nh = std::min(nh, nk);
      }
      if (nk <= nh) continue;
      c.ent_P.push_back(p);
      c.kbeg.push_back(s0 + nh);
      c.kend.push_back(s0 + nk);
      c.nquartet += nk - nh;
      c.task_off.push_back(c.task_off.back() + (nk - nh + c.KT - 1) / c.KT);
    }
  c.ntask = c.task_off.back();
  c.unit_off.clear();
  c.unit_P.clear();
  for (size_t u = 0; u < c.ent_P.size(); ++u)
    if (u == 0 || c.ent_P[u] != c.ent_P[u - 1]) {
      c.unit_off.push_back(c.task_off[u]);
      c.unit_P.push_back(c.ent_P[u]);
    }
  c.unit_off.push_back(c.ntask);
  c.usamp.assign((size_t)(c.ntask >> TASK_SAMPLE_SHIFT) + 1, 0);
  for (size_t u = 0, k = 0; k < c.usamp.size(); ++k) {
    const long long t = (long long)k << TASK_SAMPLE_SHIFT;
    while (u + 1 < c.ent_P.size() && c.task_off[u + 1] <= t) ++u;
    c.usamp[k] = (int)u;
  }
  mako_status st;
  if (c.ntask > 0 && ((st = upload(c.d_kbeg, c.kbeg)) || (st = upload(c.d_kend, c.kend)) ||
                      (st = upload(c.d_task_off, c.task_off)) || (st = upload(c.d_ent_P, c.ent_P)) ||
                      (st = upload(c.d_usamp, c.usamp)) || (st = upload(c.d_unit_off, c.unit_off)) ||
                      (st = upload(c.d_unit_P, c.unit_P))))
    return st;
  return MAKO_OK;
}

// Global task ranges [t0, t1) of shard s of n in class plan c (the interleaved chunks of shard_chunk /
// shard_task, mako_internal.h), in increasing order.
template <class F>
static void for_shard_ranges(const ClassPlan& c, int s, int n, F&& f) {
  if (c.ntask == 0) return;
  if (n == 1) { f(0LL, c.ntask); return; }
  const long long C = shard_chunk(c.ntask, n);
  for (long long j = s; j * C < c.ntask; j += n) f(j * C, std::min((j + 1) * C, c.ntask));
}

constexpr int KT_JK = 4;

// Plan for Schwarz threshold `thresh`; with tier > thresh (reduced-precision build)
// the quartets of classes that have a TF32-tier kernel are split: Q_ab Q_cd >= tier into cls (FP64),
// thresh <= Q_ab Q_cd < tier into cls_lo (TF32).  tier = 0: one FP64 tier.
static mako_status ensure_plan(mako_pairs P, double thresh, double tier = 0.0, int nshards = 1) {
  if (!(tier > thresh)) tier = 0.0;
  if (P->plan.thresh == thresh && P->plan.tier == tier && P->plan.nshards == nshards && !P->plan.cls.empty())
    return MAKO_OK;
  for (auto& sp : P->plan_cache)
    if (sp.thresh == thresh && sp.tier == tier && sp.nshards == nshards && !sp.cls.empty()) {
      std::swap(P->plan, sp);
      return MAKO_OK;
    }
  if (!P->plan.cls.empty()) {
    P->plan_cache.push_back(std::move(P->plan));
    if (P->plan_cache.size() > 6) P->plan_cache.erase(P->plan_cache.begin());
  }
  P->plan = Plan();
  Plan& pl = P->plan;
  const int NCL = NBUCKET * (NBUCKET + 1) / 2;
  pl.cls.resize(NCL);
  pl.cls_lo.resize(NCL);
  pl.KT = 16;
  const double inf = std::numeric_limits<double>::infinity();
  if (P->nsm <= 0) {
    int dev = 0;
    cudaGetDevice(&dev);
    if (cudaDeviceGetAttribute(&P->nsm, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || P->nsm <= 0) P->nsm = 148;
  }
  for (int X = 0; X < NBUCKET; ++X)
    for (int Y = 0; Y <= X; ++Y) {
      const int ci = class_index(X, Y);
      const bool split = tier > 0.0 && class_has_lowp(X, Y);
      for (int part = 0; part < (split ? 2 : 1); ++part) {
        ClassPlan& c = part ? pl.cls_lo[ci] : pl.cls[ci];
        c.X = X;
        c.Y = Y;
        c.KT = class_task_kets(X, Y);
        // warp-per-quartet classes: 4 kets per task (measured on the bench workload, tools/exp/kt.sh:
        // family time 5.60 / 5.52 / 5.47 / 5.45 s at KT = 32 / 16 / 8 / 4; the slot-batched kernel
        // batches ket primitives across the kets of a task and keeps 16)
        if (class_family(X, Y) == 4 || class_family(X, Y) == 5) c.KT = KT_JK;
        {  // experiments only (tools/exp): MAKO_KT_EXP overrides the base task length of the runtime-KT families
          static const int kt_exp = std::getenv("MAKO_KT_EXP") ? std::atoi(std::getenv("MAKO_KT_EXP")) : 0;
          const int f = class_family(X, Y);
          if (kt_exp > 0 && (f == 3 || f == 4 || f == 5)) c.KT = kt_exp;
        }
        c.swap = class_swap(X, Y);
        c.TB = c.swap ? Y : X;
        c.LB = c.swap ? X : Y;
        const double lo = part ? thresh : (split ? tier : thresh), hi = part ? tier : inf;
        mako_status st = build_class_plan(c, P->set.b[c.TB], P->set.b[c.LB], X == Y, lo, hi);
        if (st) return st;
        // warp-per-quartet and slot-batched classes (runtime KT) with few quartets (contracted or small
        // high-l workloads, e.g. the paper's E1 microbenchmark): shorter tasks so
        // that the SMs see at least ~32 grabs (TASK_GRAB tasks each) per SM instead of a few
        // long-running warps; with nshards GPUs each one sees 1/nshards of the class
        const long long want = (long long)TASK_GRAB * P->nsm * 32;
        const int fam = class_family(X, Y);
        const long long nq_shard = c.nquartet / nshards;
        if ((fam == 4 || fam == 3 || fam == 5) && nq_shard > 0 && nq_shard / c.KT < want) {
          c.KT = (int)std::max<long long>(1, nq_shard / want);
          if ((st = build_class_plan(c, P->set.b[c.TB], P->set.b[c.LB], X == Y, lo, hi))) return st;
        }
      }
    }
  pl.thresh = thresh;
  pl.tier = tier;
  pl.nshards = nshards;
  // the plan arrays were uploaded with pageable cudaMemcpy (legacy stream); the kernels that read them
  // run on non-blocking streams: wait for the DMA to land before any launch
  return cuda_check(cudaDeviceSynchronize(), "plan upload");
}

// J = Jacc + Jacc^T, K = Kacc + Kacc^T (in place)
__global__ void symmetrize_kernel(double* __restrict__ J, double* __restrict__ K, int n) {
  const long long total = (long long)n * n;
  for (long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x; x < total; x += (long long)gridDim.x * blockDim.x) {
    const int i = (int)(x / n), j = (int)(x % n);
    if (j > i) continue;
    const size_t a = (size_t)i * n + j, b = (size_t)j * n + i;
    const double sj = J[a] + J[b], sk = K[a] + K[b];
    J[a] = sj; J[b] = sj;
    K[a] = sk; K[b] = sk;
  }
}

// accumulate mode (MAKO_JK_ACCUMULATE): J += Jacc + Jacc^T, K += Kacc + Kacc^T
__global__ void symmetrize_add_kernel(const double* __restrict__ Ja, const double* __restrict__ Ka,
                                      double* __restrict__ J, double* __restrict__ K, int n) {
  const long long total = (long long)n * n;
  for (long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x; x < total; x += (long long)gridDim.x * blockDim.x) {
    const int i = (int)(x / n), j = (int)(x % n);
    const size_t a = (size_t)i * n + j, b = (size_t)j * n + i;
    J[a] += Ja[a] + Ja[b];
    K[a] += Ka[a] + Ka[b];
  }
}

// dD = D - Dprev and max |dD| (NaN-propagating, as dsh_kernel)
__global__ void delta_kernel(const double* __restrict__ D, const double* __restrict__ Dp, double* __restrict__ dD,
                             long long total, unsigned long long* __restrict__ dmax) {
  double gm = 0.0;
  for (long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x; x < total; x += (long long)gridDim.x * blockDim.x) {
    const double v = D[x] - Dp[x];
    dD[x] = v;
    const double a = fabs(v);
    gm = (a > gm || a != a) ? a : gm;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const double y = __shfl_xor_sync(0xffffffffu, gm, o);
    gm = (y > gm || y != y) ? y : gm;
  }
  if ((threadIdx.x & 31) == 0) atomicMax(dmax, (unsigned long long)__double_as_longlong(gm));
}

// density screening: dsh[sa][sb] = max |D| over the (sa, sb) block (rounded up to float); dmax = max |D|
__global__ void dsh_kernel(const double* __restrict__ D, int nbf, int nshell, const int* __restrict__ ao,
                           const int* __restrict__ l, float* __restrict__ dsh, unsigned long long* __restrict__ dmax) {
  const long long n2 = (long long)nshell * nshell;
  double gm = 0.0;
  for (long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x; x < n2; x += (long long)gridDim.x * blockDim.x) {
    const int sa = (int)(x / nshell), sb = (int)(x % nshell);
    const int oa = ao[sa], ob = ao[sb], na = 2 * l[sa] + 1, nb = 2 * l[sb] + 1;
    // NaN-propagating maxima (fmax drops NaN): a NaN anywhere in D makes dmax NaN and fails the build
    double m = 0.0;
    for (int i = 0; i < na; ++i)
      for (int j = 0; j < nb; ++j) {
        const double v = fabs(D[(size_t)(oa + i) * nbf + ob + j]);
        m = (v > m || v != v) ? v : m;
      }
    dsh[x] = __double2float_ru(m);
    gm = (m > gm || m != m) ? m : gm;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const double y = __shfl_xor_sync(0xffffffffu, gm, o);
    gm = (y > gm || y != y) ? y : gm;
  }
  // gm >= 0 or +NaN: as unsigned bit patterns these order like the values, NaN above +inf
  if ((threadIdx.x & 31) == 0) atomicMax(dmax, (unsigned long long)__double_as_longlong(gm));
}

__global__ void boys_kernel(int n, const double* __restrict__ T, double* __restrict__ out, const double* __restrict__ tab,
                            int mmax) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  double F[4 * LMAX + 1];
  switch (mmax) {
#define BCASE(m)                                                                   \
  case m: {                                                                        \
    double G[m + 1];                                                               \
    boys_eval<m>(T[i], tab, G);                                                    \
    for (int k = 0; k <= m; ++k) F[k] = G[k];                                      \
    break;                                                                         \
  }
    BCASE(0) BCASE(1) BCASE(2) BCASE(3) BCASE(4) BCASE(5) BCASE(6) BCASE(7) BCASE(8) BCASE(9) BCASE(10) BCASE(11)
    BCASE(12) BCASE(13) BCASE(14) BCASE(15) BCASE(16)
#undef BCASE
  }
  for (int k = 0; k <= mmax; ++k) out[(size_t)i * (mmax + 1) + k] = F[k];
}

}  // namespace mako

using namespace mako;

static mako_status check_pairs(mako_pairs p) {
  if (!p || !p->basis) return fail(MAKO_ERR_INVALID, "NULL pairs");
  int dev = -1;
  cudaGetDevice(&dev);
  if (dev != p->basis->device) return fail(MAKO_ERR_STATE, "pairs belong to another CUDA device");
  return MAKO_OK;
}

extern "C" mako_status mako_pairs_stats(mako_pairs p, double thresh, long long* n_pairs, long long* n_prim_pairs,
                                        long long* n_quartets) {
  try {
    mako_status st;
    if ((st = check_pairs(p))) return st;
    if (!(thresh >= 0)) return fail(MAKO_ERR_INVALID, "thresh < 0");
    thresh = std::max(thresh, p->tau);
    if ((st = ensure_plan(p, thresh))) return st;
    long long np = 0, npp = 0, nq = 0;
    for (int b = 0; b < NBUCKET; ++b) {
      np += p->set.b[b].n();
      npp += p->set.b[b].poff.back();
    }
    for (auto& c : p->plan.cls) nq += c.nquartet;
    if (n_pairs) *n_pairs = np;
    if (n_prim_pairs) *n_prim_pairs = npp;
    if (n_quartets) *n_quartets = nq;
    return MAKO_OK;
  } catch (const std::exception& e) {
    return fail(MAKO_ERR_OOM, e.what());
  }
}

// per-class algorithmic GEMM FLOPs / quartets / primitive quartets of one shard
static mako_status class_flops(mako_pairs p, double thresh, int shard, int nshards, std::vector<double>& fl,
                               std::vector<long long>& nq, std::vector<long long>& npq) {
  mako_status st;
  if ((st = check_pairs(p))) return st;
  if (!(thresh >= 0) || nshards < 1 || shard < 0 || shard >= nshards) return fail(MAKO_ERR_INVALID, "bad args");
  thresh = std::max(thresh, p->tau);
  if ((st = ensure_plan(p, thresh, 0.0, nshards))) return st;
  const int NC = NBUCKET * (NBUCKET + 1) / 2;
  fl.assign(NC, 0.0);
  nq.assign(NC, 0);
  npq.assign(NC, 0);
  for (auto& c : p->plan.cls) {
    const int KT = c.KT;
    const int ci = class_index(c.X, c.Y);
    const PairBucket& bx = p->set.b[c.TB];  // task pairs
    const PairBucket& by = p->set.b[c.LB];  // lane pairs
    // canonical orientation for the algorithmic count: bra = bucket X, ket = bucket Y
    const int la = bucket_la(c.X), lb = bucket_lb(c.X), lc = bucket_la(c.Y), ld = bucket_lb(c.Y);
    const double nab = nsph(la) * nsph(lb), ncd = nsph(lc) * nsph(ld);
    const double hab = nH(la + lb), hcd = nH(lc + ld);
    // surviving kets of each (bra, K-group) entry restricted to this shard's task ranges
    for_shard_ranges(c, shard, nshards, [&](long long t0, long long t1) {
      size_t u = std::upper_bound(c.task_off.begin(), c.task_off.end(), t0) - c.task_off.begin() - 1;
      for (; u < c.kbeg.size() && c.task_off[u] < t1; ++u) {
        const long long a0 = c.task_off[u], a1 = c.task_off[u + 1];
        if (a1 <= t0) continue;
        const int Pb = c.ent_P[u];
        const long long KAB = bx.poff[Pb + 1] - bx.poff[Pb];
        const int r0 = c.kbeg[u] + (int)(std::max(a0, t0) - a0) * KT;
        const int r1 = std::min(c.kbeg[u] + (int)(std::min(a1, t1) - a0) * KT, c.kend[u]);
        if (r1 <= r0) continue;
        const long long sumK = by.poff[r1] - by.poff[r0];
        if (!c.swap)
          fl[ci] += (double)KAB * sumK * 2.0 * nab * hab * hcd + (double)sumK * 2.0 * nab * hcd * ncd;
        else  // task pair = canonical ket (K_CD = KAB here), lanes = canonical bras (sum K_AB = sumK)
          fl[ci] += (double)KAB * sumK * 2.0 * nab * hab * hcd + (double)KAB * (r1 - r0) * 2.0 * nab * hcd * ncd;
        nq[ci] += r1 - r0;
        npq[ci] += KAB * sumK;
      }
    });
  }
  return MAKO_OK;
}

extern "C" mako_status mako_pairs_flops(mako_pairs p, double thresh, int shard, int nshards, double* gemm_flops,
                                        long long* n_quartets, long long* n_prim_quartets) {
  try {
    std::vector<double> fl;
    std::vector<long long> nq, npq;
    mako_status st = class_flops(p, thresh, shard, nshards, fl, nq, npq);
    if (st) return st;
    double f = 0;
    long long a = 0, b = 0;
    for (size_t i = 0; i < fl.size(); ++i) { f += fl[i]; a += nq[i]; b += npq[i]; }
    if (gemm_flops) *gemm_flops = f;
    if (n_quartets) *n_quartets = a;
    if (n_prim_quartets) *n_prim_quartets = b;
    return MAKO_OK;
  } catch (const std::exception& e) {
    return fail(MAKO_ERR_OOM, e.what());
  }
}

extern "C" mako_status mako_pairs_class_flops(mako_pairs p, double thresh, int shard, int nshards, double* flops,
                                              long long* quartets, long long* prim_quartets) {
  try {
    std::vector<double> fl;
    std::vector<long long> nq, npq;
    mako_status st = class_flops(p, thresh, shard, nshards, fl, nq, npq);
    if (st) return st;
    for (size_t i = 0; i < fl.size(); ++i) {
      if (flops) flops[i] = fl[i];
      if (quartets) quartets[i] = nq[i];
      if (prim_quartets) prim_quartets[i] = npq[i];
    }
    return MAKO_OK;
  } catch (const std::exception& e) {
    return fail(MAKO_ERR_OOM, e.what());
  }
}

static void drop_events(mako_pairs p) {
  for (auto& e : p->prof_events) {
    cudaEventDestroy((cudaEvent_t)e.second.first);
    cudaEventDestroy((cudaEvent_t)e.second.second);
  }
  p->prof_events.clear();
}

mako_pairs_s::~mako_pairs_s() {
  drop_events(this);
  for (void* s : streams) cudaStreamDestroy((cudaStream_t)s);
  for (void* e : ev_join) cudaEventDestroy((cudaEvent_t)e);
  if (ev_fork) cudaEventDestroy((cudaEvent_t)ev_fork);
}

// internal streams for concurrent class launches (created on first use, on the pairs' device)
static constexpr int NSTREAM = 1;  // concurrent classes measured slower (cache interference): 16.9 s vs 15.8 s
static mako_status ensure_streams(mako_pairs p) {
  if (!p->streams.empty()) return MAKO_OK;
  for (int i = 0; i < NSTREAM; ++i) {
    cudaStream_t s;
    cudaEvent_t e;
    if (cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
      return fail(MAKO_ERR_CUDA, "stream/event creation failed");
    p->streams.push_back((void*)s);
    p->ev_join.push_back((void*)e);
  }
  cudaEvent_t f;
  if (cudaEventCreateWithFlags(&f, cudaEventDisableTiming) != cudaSuccess) return fail(MAKO_ERR_CUDA, "event");
  p->ev_fork = (void*)f;
  return MAKO_OK;
}

extern "C" mako_status mako_profile_enable(mako_pairs p, int enable) {
  mako_status st;
  if ((st = check_pairs(p))) return st;
  drop_events(p);
  p->prof = enable != 0;
  return MAKO_OK;
}

extern "C" mako_status mako_profile_read(mako_pairs p, double* ms, long long* launches) {
  mako_status st;
  if ((st = check_pairs(p))) return st;
  const int NC = NBUCKET * (NBUCKET + 1) / 2;
  std::vector<double> t(NC, 0.0);
  std::vector<long long> n(NC, 0);
  for (auto& e : p->prof_events) {
    cudaError_t ce = cudaEventSynchronize((cudaEvent_t)e.second.second);
    if (ce != cudaSuccess) return cuda_check(ce, "cudaEventSynchronize");
    float x = 0.f;
    cudaEventElapsedTime(&x, (cudaEvent_t)e.second.first, (cudaEvent_t)e.second.second);
    t[e.first] += x;
    n[e.first] += 1;
  }
  for (int i = 0; i < NC; ++i) {
    if (ms) ms[i] = t[i];
    if (launches) launches[i] = n[i];
  }
  return MAKO_OK;
}

extern "C" mako_status mako_build_jk_launches(mako_pairs p, double thresh, int shard, int nshards, int* n) {
  mako_status st;
  if ((st = check_pairs(p))) return st;
  if (!n || !(thresh >= 0) || nshards < 1 || shard < 0 || shard >= nshards) return fail(MAKO_ERR_INVALID, "bad args");
  thresh = std::max(thresh, p->tau);
  if ((st = ensure_plan(p, thresh, 0.0, nshards))) return st;
  int cnt = 1;  // symmetrize
  for (auto& c : p->plan.cls)
    if (c.ntask > 0 && shard_ntask(c.ntask, shard, nshards, shard_chunk(c.ntask, nshards)) > 0) ++cnt;
  *n = cnt;
  return MAKO_OK;
}

// tier > 0 (mako_build_jk_mixed): quartets with Q_ab Q_cd max|D| >= tier stay FP64, the rest of the
// classes that have a TF32-tier kernel run it (§3.2.3)
static mako_status build_jk_impl(mako_pairs p, const double* D, double thresh, double tier, unsigned flags, double* J,
                                 double* K, int shard, int nshards, void* cuda_stream) {
  try {
    mako_status st;
    if ((st = check_pairs(p))) return st;
    if (!D || !J || !K) return fail(MAKO_ERR_INVALID, "NULL matrix");
    if (D == J || D == K || J == K) return fail(MAKO_ERR_INVALID, "D, J, K must not alias");
    if (!(thresh >= 0) || !std::isfinite(thresh)) return fail(MAKO_ERR_INVALID, "thresh must be finite and >= 0");
    if (nshards < 1 || shard < 0 || shard >= nshards) return fail(MAKO_ERR_INVALID, "shard out of range");
    if (flags & ~(unsigned)(MAKO_JK_DENSITY_SCREEN | MAKO_JK_ACCUMULATE)) return fail(MAKO_ERR_INVALID, "unknown flags");
    const mako_basis_s* B = p->basis;
    const int n = B->nbf;
    cudaStream_t s = (cudaStream_t)cuda_stream;
    if (!(tier >= 0) || !std::isfinite(tier)) return fail(MAKO_ERR_INVALID, "thresh_fp64 must be finite and >= 0");
    const bool dw = (flags & MAKO_JK_DENSITY_SCREEN) != 0;
    const double dw_thresh = std::max(thresh, p->tau);
    double tier_plan = 0.0;
    // The task counters, the D block maxima and the internal streams are per-handle state: the caller's
    // stream first waits for the previous build of this handle (which may have been enqueued on another
    // stream), so two builds in flight on one handle are serialised instead of racing on the counters.
    if ((st = ensure_streams(p))) return st;
    for (void* e : p->ev_join) cudaStreamWaitEvent(s, (cudaEvent_t)e, 0);
    if (dw || tier > 0) {
      // shell-block maxima of |D| and the global max; the task plan is the Schwarz prefix at
      // thresh / max|D| rounded down to a power of ten (a superset of the density-screened quartets,
      // few distinct plans over an SCF run), each quartet is then tested in the kernels
      const int ns = B->nshell;
      if (!p->d_dsh.p && (st = p->d_dsh.alloc(sizeof(float) * (size_t)ns * ns))) return st;
      if (!p->d_dmax.p && (st = p->d_dmax.alloc(sizeof(double)))) return st;
      if ((st = cuda_check(cudaMemsetAsync(p->d_dmax.p, 0, sizeof(double), s), "memset dmax"))) return st;
      dsh_kernel<<<592, 256, 0, s>>>(D, n, ns, B->d_ao.as<int>(), B->d_l.as<int>(), p->d_dsh.as<float>(),
                                     p->d_dmax.as<unsigned long long>());
      double dmax = 0.0;
      if ((st = cuda_check(cudaMemcpyAsync(&dmax, p->d_dmax.p, sizeof(double), cudaMemcpyDeviceToHost, s), "dmax")) ||
          (st = cuda_check(cudaStreamSynchronize(s), "dmax sync")))
        return st;
      if (!std::isfinite(dmax)) return fail(MAKO_ERR_INVALID, "D is not finite");
      if (dw) thresh = dmax > 0 ? std::pow(10.0, std::floor(std::log10(dw_thresh / dmax))) : 1e300;
      // tier boundary on Q_ab Q_cd: tier / max|D| rounded down to a power of ten (more FP64 work, few
      // distinct plans over an SCF run)
      if (tier > 0) tier_plan = dmax > 0 ? std::pow(10.0, std::floor(std::log10(tier / dmax))) : 0.0;
    }
    thresh = std::max(thresh, p->tau);
    if ((st = ensure_plan(p, thresh, tier_plan, nshards))) return st;
    const bool mixed = p->plan.tier > 0.0;
    if (mixed && (st = ensure_lowp(p->set, cuda_stream))) return st;
    // accumulate mode: the kernels fill per-handle scratch accumulators, added into J/K at the end
    const bool acc = (flags & MAKO_JK_ACCUMULATE) != 0;
    const size_t n2 = (size_t)n * n;
    if (acc && !p->d_jk_scratch.p && (st = p->d_jk_scratch.alloc(2 * sizeof(double) * n2))) return st;
    double* Jw = acc ? p->d_jk_scratch.as<double>() : J;
    double* Kw = acc ? p->d_jk_scratch.as<double>() + n2 : K;
    if ((st = cuda_check(cudaMemsetAsync(Jw, 0, sizeof(double) * n2, s), "memset J")) ||
        (st = cuda_check(cudaMemsetAsync(Kw, 0, sizeof(double) * n2, s), "memset K")) ||
        (st = cuda_check(cudaMemsetAsync(p->d_counters.p, 0, sizeof(unsigned long long) * 2 * NCLASS, s), "memset ctr")))
      return st;
    int nl = 0;
    // fork: internal streams wait for the zeroed J/K on the caller's stream
    cudaEventRecord((cudaEvent_t)p->ev_fork, s);
    for (void* is : p->streams) cudaStreamWaitEvent((cudaStream_t)is, (cudaEvent_t)p->ev_fork, 0);
    // classes in descending estimated cost, greedily balanced over the internal streams; each kernel
    // gets half of the resident capacity so two classes (often a DFMA- and a DMMA-bound one) co-reside
    // (index >= NCLASS: the class's TF32-tier plan)
    const int NCL = (int)p->plan.cls.size();
    std::vector<std::pair<double, int>> order;
    for (int i = 0; i < (mixed ? 2 * NCL : NCL); ++i) {
      const ClassPlan& c = i < NCL ? p->plan.cls[i] : p->plan.cls_lo[i - NCL];
      if (c.ntask == 0) continue;
      const double cost = (double)c.nquartet * (nsph(bucket_la(c.X)) * nsph(bucket_lb(c.X)) *
                                                    nsph(bucket_la(c.Y)) * nsph(bucket_lb(c.Y)) + 16.0);
      order.push_back({-cost, i});
    }
    std::sort(order.begin(), order.end());
    std::vector<double> load(p->streams.size(), 0.0);
    for (auto& oc : order) {
      const bool lo = oc.second >= NCL;
      ClassPlan& c = lo ? p->plan.cls_lo[oc.second - NCL] : p->plan.cls[oc.second];
      JKArgs a{};
      a.ntask = c.ntask;
      a.shard = shard;
      a.nshards = nshards;
      a.chunk = nshards == 1 ? c.ntask : shard_chunk(c.ntask, nshards);
      a.ntask_local = nshards == 1 ? c.ntask : shard_ntask(c.ntask, shard, nshards, a.chunk);
      if (a.ntask_local <= 0) continue;
      const size_t si = std::min_element(load.begin(), load.end()) - load.begin();
      load[si] += -oc.first;
      cudaStream_t cs = (cudaStream_t)p->streams[si];
      a.bra = p->set.b[c.TB].view();
      a.ket = p->set.b[c.LB].view();
      a.same_bucket = c.X == c.Y;
      a.task_off = c.d_task_off.as<long long>();
      a.kbeg = c.d_kbeg.as<int>();
      a.kend = c.d_kend.as<int>();
      a.ent_P = c.d_ent_P.as<int>();
      a.usamp = c.d_usamp.as<int>();
      a.nent = (int)c.kbeg.size();
      a.nunit = (int)c.unit_P.size();
      a.unit_off = c.d_unit_off.as<long long>();
      a.unit_P = c.d_unit_P.as<int>();
      a.shl = B->d_l.as<int>();
      a.KT = c.KT;
      a.counter = p->d_counters.as<unsigned long long>() + class_index(c.X, c.Y) + (lo ? NCL : 0);
      a.D = D;
      a.J = Jw;
      a.K = Kw;
      a.nbf = n;
      a.ao = B->d_ao.as<int>();
      a.thresh = thresh;
      a.dsh = dw ? p->d_dsh.as<float>() : nullptr;
      a.nshell = B->nshell;
      a.dw_thresh = dw_thresh;
      a.boys = B->d_boys.as<double>();
      a.grid_div = 1;
      a.lowp = lo ? 1 : 0;
      cudaEvent_t e0 = nullptr, e1 = nullptr;
      if (p->prof) {
        cudaEventCreate(&e0);
        cudaEventCreate(&e1);
        cudaEventRecord(e0, cs);
      }
      if ((st = launch_jk_class(c.X, c.Y, a, (void*)cs, &nl))) return st;
      if (p->prof) {
        cudaEventRecord(e1, cs);
        p->prof_events.push_back({class_index(c.X, c.Y), {(void*)e0, (void*)e1}});
      }
    }
    // join: the caller's stream waits for every internal stream
    for (size_t i = 0; i < p->streams.size(); ++i) {
      cudaEventRecord((cudaEvent_t)p->ev_join[i], (cudaStream_t)p->streams[i]);
      cudaStreamWaitEvent(s, (cudaEvent_t)p->ev_join[i], 0);
    }
    if (acc) symmetrize_add_kernel<<<592, 256, 0, s>>>(Jw, Kw, J, K, n);
    else symmetrize_kernel<<<592, 256, 0, s>>>(J, K, n);
    return cuda_check(cudaGetLastError(), "symmetrize launch");
  } catch (const std::exception& e) {
    return fail(MAKO_ERR_OOM, e.what());
  }
}

extern "C" mako_status mako_build_jk(mako_pairs p, const double* D, double thresh, double* J, double* K, int shard,
                                     int nshards, void* cuda_stream) {
  return build_jk_impl(p, D, thresh, 0.0, 0u, J, K, shard, nshards, cuda_stream);
}

extern "C" mako_status mako_build_jk_ex(mako_pairs p, const double* D, double thresh, unsigned flags, double* J,
                                        double* K, int shard, int nshards, void* cuda_stream) {
  return build_jk_impl(p, D, thresh, 0.0, flags, J, K, shard, nshards, cuda_stream);
}

extern "C" mako_status mako_build_jk_mixed(mako_pairs p, const double* D, double thresh, double thresh_fp64,
                                           unsigned flags, double* J, double* K, int shard, int nshards,
                                           void* cuda_stream) {
  if (!(thresh_fp64 > 0) || !std::isfinite(thresh_fp64)) return fail(MAKO_ERR_INVALID, "thresh_fp64 must be > 0");
  return build_jk_impl(p, D, thresh, thresh_fp64, flags, J, K, shard, nshards, cuda_stream);
}

extern "C" mako_status mako_density_delta(mako_pairs p, const double* D, const double* D_prev, double* dD,
                                          double* dmax, void* cuda_stream) {
  try {
    mako_status st;
    if ((st = check_pairs(p))) return st;
    if (!D || !D_prev || !dD || !dmax) return fail(MAKO_ERR_INVALID, "NULL argument");
    if (dD == D || dD == D_prev) return fail(MAKO_ERR_INVALID, "dD must not alias D or D_prev");
    const int n = p->basis->nbf;
    cudaStream_t s = (cudaStream_t)cuda_stream;
    if (!p->d_dmax.p && (st = p->d_dmax.alloc(sizeof(double)))) return st;
    if ((st = ensure_streams(p))) return st;
    for (void* e : p->ev_join) cudaStreamWaitEvent(s, (cudaEvent_t)e, 0);  // d_dmax is per-handle state
    if ((st = cuda_check(cudaMemsetAsync(p->d_dmax.p, 0, sizeof(double), s), "memset dmax"))) return st;
    delta_kernel<<<592, 256, 0, s>>>(D, D_prev, dD, (long long)n * n, p->d_dmax.as<unsigned long long>());
    double h = 0.0;
    if ((st = cuda_check(cudaMemcpyAsync(&h, p->d_dmax.p, sizeof(double), cudaMemcpyDeviceToHost, s), "dmax")) ||
        (st = cuda_check(cudaStreamSynchronize(s), "delta sync")))
      return st;
    *dmax = h;
    if (!std::isfinite(h)) return fail(MAKO_ERR_INVALID, "D or D_prev is not finite");
    return MAKO_OK;
  } catch (const std::exception& e) {
    return fail(MAKO_ERR_OOM, e.what());
  }
}

extern "C" mako_status mako_class_family(int* family) {
  if (!family) return fail(MAKO_ERR_INVALID, "NULL family");
  for (int X = 0; X < NBUCKET; ++X)
    for (int Y = 0; Y <= X; ++Y) family[class_index(X, Y)] = class_family(X, Y);
  return MAKO_OK;
}

extern "C" mako_status mako_class_reduced(int* mask) {
  if (!mask) return fail(MAKO_ERR_INVALID, "NULL mask");
  for (int X = 0; X < NBUCKET; ++X)
    for (int Y = 0; Y <= X; ++Y) mask[class_index(X, Y)] = class_has_lowp(X, Y) ? 1 : 0;
  return MAKO_OK;
}

static mako_status eri_batch_impl(mako_basis basis, int nq, const int* quartets, double* out, size_t out_len,
                                  unsigned flags, void* cuda_stream) {
  try {
    if (flags & ~(unsigned)MAKO_ERI_REDUCED) return fail(MAKO_ERR_INVALID, "unknown flags");
    if (!basis || (nq > 0 && (!quartets || !out))) return fail(MAKO_ERR_INVALID, "NULL argument");
    if (nq < 0) return fail(MAKO_ERR_INVALID, "nq < 0");
    int dev = -1;
    cudaGetDevice(&dev);
    if (dev != basis->device) return fail(MAKO_ERR_STATE, "basis belongs to another CUDA device");
    size_t total = 0;
    for (int q = 0; q < nq; ++q) {
      size_t sz = 1;
      for (int k = 0; k < 4; ++k) {
        int sh = quartets[4 * q + k];
        if (sh < 0 || sh >= basis->nshell) return fail(MAKO_ERR_INVALID, "shell index out of range");
        sz *= nsph(basis->l[sh]);
      }
      total += sz;
    }
    if (total != out_len) return fail(MAKO_ERR_INVALID, "out_len does not match the total block size");
    if (nq == 0) return MAKO_OK;
    // canonicalise; one temporary pair per (bra or ket) occurrence
    std::vector<int> A[NBUCKET], Bs[NBUCKET];
    struct Item { int X, Y, P, R, flag; long long off; };
    std::vector<Item> items(nq);
    size_t off = 0;
    for (int q = 0; q < nq; ++q) {
      int u[4] = {quartets[4 * q], quartets[4 * q + 1], quartets[4 * q + 2], quartets[4 * q + 3]};
      int flag = 0;
      int ba = u[0], bb = u[1], ka = u[2], kb = u[3];
      if (basis->l[ba] < basis->l[bb]) { std::swap(ba, bb); flag |= 1; }
      if (basis->l[ka] < basis->l[kb]) { std::swap(ka, kb); flag |= 2; }
      int X = bucket_of(basis->l[ba], basis->l[bb]), Y = bucket_of(basis->l[ka], basis->l[kb]);
      if (X < Y) { std::swap(ba, ka); std::swap(bb, kb); std::swap(X, Y); flag |= 4; }
      Item& it = items[q];
      it.X = X; it.Y = Y; it.flag = flag; it.off = (long long)off;
      it.P = (int)A[X].size(); A[X].push_back(ba); Bs[X].push_back(bb);
      it.R = (int)A[Y].size(); A[Y].push_back(ka); Bs[Y].push_back(kb);
      size_t sz = 1;
      for (int k = 0; k < 4; ++k) sz *= nsph(basis->l[u[k]]);
      off += sz;
    }
    PairSet set;
    mako_status st;
    if ((st = build_pair_set(basis, A, Bs, set, cuda_stream))) return st;
    const bool lowp = (flags & MAKO_ERI_REDUCED) != 0;
    if (lowp && (st = ensure_lowp(set, cuda_stream))) return st;
    cudaStream_t s = (cudaStream_t)cuda_stream;
    std::vector<std::unique_ptr<DevBuf>> keep;
    for (int X = 0; X < NBUCKET; ++X)
      for (int Y = 0; Y <= X; ++Y) {
        std::vector<int> qb, qk, qf;
        std::vector<long long> qo;
        for (auto& it : items)
          if (it.X == X && it.Y == Y) { qb.push_back(it.P); qk.push_back(it.R); qf.push_back(it.flag); qo.push_back(it.off); }
        if (qb.empty()) continue;
        for (int k = 0; k < 4; ++k) keep.emplace_back(new DevBuf);
        DevBuf& d1 = *keep[keep.size() - 4];
        DevBuf& d2 = *keep[keep.size() - 3];
        DevBuf& d3 = *keep[keep.size() - 2];
        DevBuf& d4 = *keep[keep.size() - 1];
        if ((st = upload_async(d1, qb, s)) || (st = upload_async(d2, qk, s)) || (st = upload_async(d3, qf, s)) ||
            (st = upload_async(d4, qo, s)))
          return st;
        BatchArgs a{};
        a.bra = set.b[X].view();
        a.ket = set.b[Y].view();
        a.nq = (int)qb.size();
        a.qbra = d1.as<int>(); a.qket = d2.as<int>(); a.qflag = d3.as<int>(); a.qout = d4.as<long long>();
        a.out = out;
        a.boys = basis->d_boys.as<double>();
        a.diag = 0;
        a.lowp = lowp ? 1 : 0;
        if ((st = launch_batch_class(X, Y, a, cuda_stream))) return st;
      }
    return cuda_check(cudaStreamSynchronize(s), "eri_batch sync");
  } catch (const std::exception& e) {
    return fail(MAKO_ERR_OOM, e.what());
  }
}

extern "C" mako_status mako_eri_batch(mako_basis basis, int nq, const int* quartets, double* out, size_t out_len,
                                      void* cuda_stream) {
  return eri_batch_impl(basis, nq, quartets, out, out_len, 0u, cuda_stream);
}

extern "C" mako_status mako_eri_batch_ex(mako_basis basis, int nq, const int* quartets, double* out, size_t out_len,
                                         unsigned flags, void* cuda_stream) {
  return eri_batch_impl(basis, nq, quartets, out, out_len, flags, cuda_stream);
}

extern "C" mako_status mako_boys(int n, const double* T, int mmax, double* out, void* cuda_stream) {
  if (n < 0 || (n > 0 && (!T || !out)) || mmax < 0 || mmax > 4 * LMAX) return fail(MAKO_ERR_INVALID, "bad args");
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) return fail(MAKO_ERR_CUDA, "no CUDA device");
  if (n == 0) return MAKO_OK;
  static DevBuf tab;
  static int tab_dev = -1;
  int dev = 0;
  cudaGetDevice(&dev);
  if (tab_dev != dev) {
    std::vector<double> h;
    boys_table(h);
    mako_status st = upload(tab, h);
    if (st) return st;
    if ((st = cuda_check(cudaDeviceSynchronize(), "boys table upload"))) return st;
    tab_dev = dev;
  }
  boys_kernel<<<(n + 127) / 128, 128, 0, (cudaStream_t)cuda_stream>>>(n, T, out, tab.as<double>(), mmax);
  return cuda_check(cudaGetLastError(), "boys launch");
}
