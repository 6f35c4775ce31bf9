// eri_core.cuh -- per-class McMurchie-Davidson ERI machinery for sm_100a (FP64, DMMA).
//
// One warp evaluates one shell quartet (ab|cd) of class (la lb|lc ld) as the matrix-shaped
// stages of PAPER.md Alg. 1 (L194-L213):
//   a4 Boys F_m(T)              PAPER.md:L173-L177 (Taylor grid + downward recursion, reading R1)
//   a5 R-tensor, Eq. 5          PAPER.md:L179-L180, warp-cooperative, level by level in SMEM
//   a6 [p|q] = (-1)^{l_q}[p+q]  PAPER.md:L182-L184, gathered straight into DMMA B fragments through
//                               an index table (the paper's SL->BL "transpose", L233-L249, without
//                               materialising [p|q]); the sign is folded into E~_CD
//   a7 GEMM1 [ab|q] += E~_AB [p|q]      PAPER.md:L186-L188 Eq. 7, mma.sync.m8n8k4.f64 (DMMA)
//   a8 GEMM2 (ab|cd) += [ab|q] E~_CD^T  Eq. 7 / Eq. 11 (L251-L271), chained in registers: the
//                               m8n8 accumulator of GEMM1 IS the A operand of GEMM2 (no SMEM trip)
//   a9 digestion into FP64 J/K  (north_star; L296 FP64 accumulation)
// The spherical transform, contraction coefficients and 1/p are folded into E~ (pairs.cu).
#pragma once

#include <cuda_runtime.h>

#include "mako_internal.h"

namespace mako {

constexpr double TWO_PI_52 = 34.98683665524972497;  // 2 pi^{5/2}
constexpr double PI_D = 3.14159265358979323846;

MK_HD constexpr int clampi(int v, int lo, int hi) { return v < lo ? lo : (v > hi ? hi : v); }
MK_HD constexpr int bla(int b) { return b_la(b); }
MK_HD constexpr int blb(int b) { return b - bla(b) * (bla(b) + 1) / 2; }

template <int LA_, int LB_, int LC_, int LD_>
struct Cls {
  static constexpr int LA = LA_, LB = LB_, LC = LC_, LD = LD_;
  static constexpr int LAB = LA + LB, LCD = LC + LD, L = LAB + LCD;
  static constexpr int NA = 2 * LA + 1, NB = 2 * LB + 1, NC = 2 * LC + 1, ND = 2 * LD + 1;
  static constexpr int NAB = NA * NB, NCD = NC * ND;
  static constexpr int NHAB = nH(LAB), NHCD = nH(LCD), NH = nH(L);
  static constexpr int MT = (NAB + 7) / 8;    // m8 tiles over ab
  static constexpr int NT1 = (NHCD + 7) / 8;  // GEMM1 n8 tiles over q
  static constexpr int KS1 = (NHAB + 3) / 4;  // GEMM1 k4 steps over p
  static constexpr int NT2 = (NCD + 7) / 8;   // GEMM2 n8 tiles over cd
  // register budget for the accumulators (doubles per lane): MC m-tiles per chunk
#ifndef MAKO_REGB_HI
#define MAKO_REGB_HI 56
#endif
#ifndef MAKO_REGB_LO
#define MAKO_REGB_LO 40
#endif
  static constexpr int REGB = L >= 8 ? MAKO_REGB_HI : MAKO_REGB_LO;
  static constexpr int MCMAX = clampi(REGB / (2 * (NT1 + NT2)), 1, MT);
  static constexpr int NCHUNK = (MT + MCMAX - 1) / MCMAX;
  static constexpr int MC = (MT + NCHUNK - 1) / NCHUNK;
  // per-warp shared memory (doubles)
  // R rows kept per bra primitive (computed once per primitive quartet, reused by every row chunk)
  // (d/f x d/f bra pairs are single-primitive in the def2/cc families: no rows to group)
  static constexpr int KR = (LA >= 2 && LB >= 2) ? 1 : clampi(1200 / NH - 1, 1, 4);
  // batched R (quartet_block_rb): the R rows of up to RB primitive quartets (ket primitive x all bra
  // primitives) are computed lane-per-quartet in registers (r_regs) and stored at the odd stride RS
  static constexpr bool RBATCH = L <= 6 && in_list(kRBatchPick, bucket_of(LA, LB) * 100 + bucket_of(LC, LD));
  static constexpr int RB = 16, RS = NH | 1;
  static constexpr int W_RBAT = RBATCH ? RB * RS : 0;
  static constexpr int W_RCOOP = (KR + 1) * NH > W_RBAT ? (KR + 1) * NH : W_RBAT;
  // GEMM2 B operands from the fragment-order copy (default) or the row-major E~ (classes measured faster
  // that way, MAKO_NOFRAGB_PICK; S6)
  static constexpr bool FRAGB = !in_list(kNoFragBPick, bucket_of(LA, LB) * 100 + bucket_of(LC, LD));
  // KR result rows + 1 ping-pong scratch row; doubles as the digestion partial-sum scratch (Ps)
  static constexpr int W_R = (W_RCOOP > 2 * (NA + NB) * NCD) ? W_RCOOP : 2 * (NA + NB) * NCD;
  static constexpr int W_V = NAB * NCD; // (ab|cd) block
  static constexpr int W_J = NAB;       // J_ab partial sums over the kets of a task
  static constexpr int W_D = NA * NB + NC * ND + NA * NC + NA * ND + NB * NC + NB * ND;  // staged D blocks
  static constexpr int WARP_DBL = W_R + W_V + W_J + W_D;
  // CTA tables
  static constexpr int HTAB_BYTES = ((NHAB * NHCD * 2 + 15) / 16) * 16;
  static constexpr int RTAB_BYTES = ((NH * 4 + 15) / 16) * 16;
};

template <int X, int Y>
using ClsXY = Cls<bla(X), blb(X), bla(Y), blb(Y)>;

// ---------------------------------------------------------------------------
MK_HD inline void hdecode(int e, int& t, int& u, int& v) {
  int k = 0;
  while (nH(k) <= e) ++k;
  int r = e - nH(k - 1);
  int s = 0;
  while ((s + 1) * (s + 2) / 2 <= r) ++s;
  v = r - s * (s + 1) / 2;
  u = s - v;
  t = k - s;
}

// [pc][qc] -> Hermite index of p+q ; rtab[e] = packed recursion step for Hermite entry e
template <class C>
__device__ void init_tables(uint16_t* htab, uint32_t* rtab) {
  for (int o = threadIdx.x; o < C::NHAB * C::NHCD; o += blockDim.x) {
    int p = o / C::NHCD, q = o % C::NHCD, t1, u1, v1, t2, u2, v2;
    hdecode(p, t1, u1, v1);
    hdecode(q, t2, u2, v2);
    htab[o] = (uint16_t)hidx(t1 + t2, u1 + u2, v1 + v2);
  }
  for (int e = threadIdx.x; e < C::NH; e += blockDim.x) {
    uint32_t w = 0;
    if (e > 0) {
      int tt, uu, vv;
      hdecode(e, tt, uu, vv);
      int dir = tt > 0 ? 0 : (uu > 0 ? 1 : 2);
      int n = dir == 0 ? tt : (dir == 1 ? uu : vv);
      int s1 = dir == 0 ? hidx(tt - 1, uu, vv) : (dir == 1 ? hidx(tt, uu - 1, vv) : hidx(tt, uu, vv - 1));
      int s2 = 0;
      if (n >= 2) s2 = dir == 0 ? hidx(tt - 2, uu, vv) : (dir == 1 ? hidx(tt, uu - 2, vv) : hidx(tt, uu, vv - 2));
      w = (uint32_t)s1 | ((uint32_t)s2 << 10) | ((uint32_t)dir << 20) | ((uint32_t)(n - 1) << 22);
    }
    rtab[e] = w;
  }
}

// 256-bit read-only global load (sm_100a LDG.E.ENL2.256): 4 doubles from a 32 B aligned address
__device__ __forceinline__ void ldg256(const double* __restrict__ p, double& a, double& b, double& c, double& d) {
  asm("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];" : "=d"(a), "=d"(b), "=d"(c), "=d"(d) : "l"(p));
}

// asynchronous 8-byte global -> shared copy (LDGSTS, no register staging) and its completion wait
__device__ __forceinline__ void cp_async8(double* smem_dst, const double* gsrc) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(smem_dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(d), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;\n" ::: "memory"); }

// 1/sqrt(x) for positive normal x: float seed + two Newton steps (no slow path)
__device__ __forceinline__ double rsqrt_fast(double x) {
  double y = (double)rsqrtf((float)x);
  const double h = 0.5 * x;
  y = y * fma(-h * y, y, 1.5);
  y = y * fma(-h * y, y, 1.5);
  return y;
}

// Boys F_m(T), m = 0..L (PAPER.md:L177 lookup-table evaluation; accuracy contract: reading R1).
//  T < 40:  7-term Taylor expansion of F_L about the nearest grid point T_k = k/32 (|x| <= 1/64),
//           exp(-T) = exp(-T_k) * sum_j x^j/j! from the same row, then the exact downward
//           recursion F_m = (2T F_{m+1} + e^{-T}) / (2m+1).
//  T >= 40: F_0 = (1/2) sqrt(pi/T) (erfc(sqrt 40) < 1e-18), upward F_{m+1} = ((2m+1)F_m - e^{-T})/(2T)
//           with exp(-T) from a second 1/32 grid for T < 80 and dropped beyond (< 1e-18 relative).
// WIDE: 256-bit row loads (lane-private lookups, per-lane kernels); otherwise 128-bit loads (the
// warp-uniform lookups of the warp-cooperative R, measured faster with the narrower form)
template <int L, bool WIDE = false>
__device__ __forceinline__ void boys_eval(double T, const double* __restrict__ tab, double (&F)[L + 1]) {
  if (T < BOYS_TMAX) {
    const int k = __double2int_rn(T * (1.0 / BOYS_H));
    const double x = fma((double)k, BOYS_H, -T);
    const double* r = tab + ((size_t)L * BOYS_NGRID + k) * BOYS_ROW;  // 64 B row
    double2 r01, r23, r45, r6e;
    if constexpr (WIDE) {
      ldg256(r, r01.x, r01.y, r23.x, r23.y);
      ldg256(r + 4, r45.x, r45.y, r6e.x, r6e.y);
    } else {
      const double2* r2 = reinterpret_cast<const double2*>(r);
      r01 = __ldg(r2); r23 = __ldg(r2 + 1); r45 = __ldg(r2 + 2); r6e = __ldg(r2 + 3);
    }
    const double x2 = x * 0.5, x3 = x * (1.0 / 3.0), x4 = x * 0.25, x5 = x * 0.2, x6 = x * (1.0 / 6.0);
    double f = r6e.x;
    f = fma(f, x6, r45.y);
    f = fma(f, x5, r45.x);
    f = fma(f, x4, r23.y);
    f = fma(f, x3, r23.x);
    f = fma(f, x2, r01.y);
    f = fma(f, x, r01.x);
    F[L] = f;
    if constexpr (L > 0) {
      double e = fma(x6, 1.0, 1.0);
      e = fma(e, x5, 1.0);
      e = fma(e, x4, 1.0);
      e = fma(e, x3, 1.0);
      e = fma(e, x2, 1.0);
      e = fma(e, x, 1.0);
      e *= r6e.y;
      const double t2 = 2.0 * T;
#pragma unroll
      for (int m = L - 1; m >= 0; --m) F[m] = fma(t2, F[m + 1], e) * (1.0 / (2 * m + 1));
    }
  } else {
    const double rs = rsqrt_fast(T);
    F[0] = 0.88622692545275801365 * rs;  // sqrt(pi)/2
    if constexpr (L > 0) {
      double e = 0.0;
      if (T < BOYS_TEXP) {
        const int k = __double2int_rn((T - BOYS_TMAX) * (1.0 / BOYS_H));
        const double x = fma((double)k, BOYS_H, BOYS_TMAX - T);
        double s = fma(x, 1.0 / 6.0, 1.0);
        s = fma(s, x * 0.2, 1.0);
        s = fma(s, x * 0.25, 1.0);
        s = fma(s, x * (1.0 / 3.0), 1.0);
        s = fma(s, x * 0.5, 1.0);
        s = fma(s, x, 1.0);
        e = s * __ldg(tab + BOYS_EXP_OFF + k);
      }
      const double h = 0.5 * rs * rs;
#pragma unroll
      for (int m = 0; m < L; ++m) F[m + 1] = fma((double)(2 * m + 1), F[m], -e) * h;
    }
  }
}

// R^{(0)}_{tuv}(rho, P-Q) for t+u+v <= L into buf[0..NH) (Eq. 4-5):
//   R^{(n)}_{000} = (-2 rho)^n F_n(rho |PQ|^2) * 2 pi^{5/2} / sqrt(p+q)
//   R^{(n)}_{t+1,u,v} = t R^{(n+1)}_{t-1,u,v} + X_PQ R^{(n+1)}_{t,u,v}   (and u, v alike)
// Level n holds all entries with t+u+v <= L-n; lanes split each level; levels ping-pong.
// F32: level 0 is written TF32-rounded into dst32 instead of dst (reduced-precision tier, eri_quant.cuh;
// the recursion itself stays FP64)
__device__ __forceinline__ float to_tf32(double x) {
  unsigned r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"((float)x));
  return __uint_as_float(r);
}

template <class C, bool F32 = false>
__device__ __forceinline__ void compute_R(double p, double Px, double Py, double Pz, double q, double Qx, double Qy,
                                          double Qz, double* __restrict__ dst, double* __restrict__ scratch,
                                          const uint32_t* __restrict__ rtab, const double* __restrict__ btab,
                                          int lane, float* __restrict__ dst32 = nullptr) {
  constexpr int L = C::L, NH = C::NH;
  const double pq = p + q, ri = rsqrt_fast(pq), rho = p * q * ri * ri;
  const double X = Px - Qx, Y = Py - Qy, Z = Pz - Qz;
  const double T = rho * (X * X + Y * Y + Z * Z);
  double F[L + 1];
  boys_eval<L>(T, btab, F);
  double s = TWO_PI_52 * ri;
  const double m2r = -2.0 * rho;
#pragma unroll
  for (int n = 0; n <= L; ++n) {
    F[n] *= s;
    s *= m2r;
  }
  if constexpr (L == 0) {
    if (lane == 0) {
      if constexpr (F32) dst32[0] = to_tf32(F[0]);
      else dst[0] = F[0];
    }
    __syncwarp();
  } else {
    if (lane == 0) ((L & 1) ? scratch : dst)[0] = F[L];
    __syncwarp();
#pragma unroll
    for (int n = L - 1; n >= 0; --n) {
      double* cur = (n & 1) ? scratch : dst;  // level 0 lands in dst
      const double* prv = ((n + 1) & 1) ? scratch : dst;
      const int cnt = nH(L - n);
#ifndef MAKO_R_ILP_LMAX
#define MAKO_R_ILP_LMAX 7
#endif
      if constexpr (L > MAKO_R_ILP_LMAX) {  // high-l classes: measured faster with one entry in flight
      for (int e = lane; e < cnt; e += 32) {
        double v;
        if (e == 0) {
          v = F[n];
        } else {
          const uint32_t w = rtab[e];
          const int s1 = w & 1023, s2 = (w >> 10) & 1023, dir = (w >> 20) & 3, cf = (int)(w >> 22);
          const double xd = dir == 0 ? X : (dir == 1 ? Y : Z);
          v = xd * prv[s1];
          if (cf) v = fma((double)cf, prv[s2], v);
        }
        if (F32 && n == 0) dst32[e] = to_tf32(v);
        else cur[e] = v;
      }
      } else {
      // up to RB entries per lane in flight: all their rtab / prv loads are issued before the first
      // store (the level loop is latency-bound on the SMEM round trips, profiles/README.md)
      constexpr int RB = 4;
      const int nj = (cnt + 31) >> 5;
#pragma unroll
      for (int j0 = 0; j0 < nj; j0 += RB) {
        double v[RB];
#pragma unroll
        for (int jj = 0; jj < RB; ++jj) {
          const int e = lane + 32 * (j0 + jj);
          v[jj] = 0.0;
          if (j0 + jj < nj && e < cnt) {
            if (e == 0) {
              v[jj] = F[n];
            } else {
              const uint32_t w = rtab[e];
              const int s1 = w & 1023, s2 = (w >> 10) & 1023, dir = (w >> 20) & 3, cf = (int)(w >> 22);
              const double xd = dir == 0 ? X : (dir == 1 ? Y : Z);
              double t = xd * prv[s1];
              if (cf) t = fma((double)cf, prv[s2], t);
              v[jj] = t;
            }
          }
        }
#pragma unroll
        for (int jj = 0; jj < RB; ++jj) {
          const int e = lane + 32 * (j0 + jj);
          if (j0 + jj < nj && e < cnt) {
            if (F32 && n == 0) dst32[e] = to_tf32(v[jj]);
            else cur[e] = v[jj];
          }
        }
      }
      }
      __syncwarp();
    }
  }
}

// primitive-pair record {p, Px, Py, Pz} (32 B aligned): one 256-bit load (WIDE) or two 128-bit loads
template <bool WIDE = false>
__device__ __forceinline__ void load_pdat(const double* __restrict__ pdat, int i, double& p, double& x, double& y,
                                          double& z) {
  if constexpr (WIDE) {
    ldg256(pdat + 4 * (size_t)i, p, x, y, z);
  } else {
    const double2* v = reinterpret_cast<const double2*>(pdat + 4 * (size_t)i);
    const double2 a = __ldg(v), b = __ldg(v + 1);
    p = a.x; x = a.y; y = b.x; z = b.y;
  }
}

__device__ __forceinline__ void dmma884(double& c0, double& c1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
               : "+d"(c0), "+d"(c1)
               : "d"(a), "d"(b));
}

// GEMM1 A operands from the fragment-order copy (MAKO_FRAG_A, default) or the row-major E~ (experiment
// switch); the GEMM2 B operand choice is per class (Cls::FRAGB)
#ifndef MAKO_FRAG_A
#define MAKO_FRAG_A 1
#endif
template <class C>
__device__ __forceinline__ const double* ebra_ptr(const PairView& bra, int ij) {
  if constexpr (MAKO_FRAG_A) return bra.EbraD + (size_t)ij * frag_a_doubles(C::LA, C::LB);
  else return bra.Ebra + (size_t)ij * (C::NAB * C::NHAB);
}

// GEMM1 k-loop of one R row (Eq. 7a): t1[mc][nt] += E~_ab[row chunk ch][p] [p|q]; the A fragments come
// from the fragment-order copy EA = EbraD + ij * frag_a_doubles (one coalesced warp load each), the B
// fragment is gathered from the R row through htab (a6)
template <class C>
__device__ __forceinline__ void gemm1_row(double (&t1)[C::MC][C::NT1][2], const double* __restrict__ EA,
                                          const double* __restrict__ Rr, const uint16_t* __restrict__ htab, int ch,
                                          int lane) {
  const int g = lane >> 2, t = lane & 3;
#pragma unroll
  for (int ks = 0; ks < C::KS1; ++ks) {
    const int pc = 4 * ks + t;
    double a[C::MC];
#pragma unroll
    for (int mc = 0; mc < C::MC; ++mc) {
      if constexpr (MAKO_FRAG_A) {
        a[mc] = (ch * C::MC + mc < C::MT) ? __ldg(EA + ((ch * C::MC + mc) * C::KS1 + ks) * 32 + lane) : 0.0;
      } else {  // EA = row-major E~_ab of the primitive pair
        const int row = 8 * (ch * C::MC + mc) + g;
        a[mc] = (row < C::NAB && pc < C::NHAB) ? __ldg(EA + row * C::NHAB + pc) : 0.0;
      }
    }
#pragma unroll
    for (int nt = 0; nt < C::NT1; ++nt) {
      const int qc = 8 * nt + g;
      const double b = (pc < C::NHAB && qc < C::NHCD) ? Rr[htab[pc * C::NHCD + qc]] : 0.0;
#pragma unroll
      for (int mc = 0; mc < C::MC; ++mc)
        if (ch * C::MC + mc < C::MT) dmma884(t1[mc][nt][0], t1[mc][nt][1], a[mc], b);
    }
  }
}

// GEMM2 (Eq. 7b / Eq. 11) chained in registers: k-step (nt, e) takes q = 8 nt + 2 t + e from the
// GEMM1 accumulator of lane (g, t); both B fragments of (nt, e = 0, 1) come with one 128-bit load from
// the fragment-order copy EB = EketD + kl * frag_b_doubles
template <class C>
__device__ __forceinline__ void gemm2_chain(double (&c2)[C::MC][C::NT2][2], const double (&t1)[C::MC][C::NT1][2],
                                            const double* __restrict__ EB, int ch, int lane) {
  if constexpr (C::FRAGB) {
#pragma unroll
    for (int nt = 0; nt < C::NT1; ++nt) {
      double2 b[C::NT2];
#pragma unroll
      for (int n2 = 0; n2 < C::NT2; ++n2) b[n2] = __ldg(reinterpret_cast<const double2*>(EB) + (nt * C::NT2 + n2) * 32 + lane);
#pragma unroll
      for (int e = 0; e < 2; ++e)
#pragma unroll
        for (int n2 = 0; n2 < C::NT2; ++n2)
#pragma unroll
          for (int mc = 0; mc < C::MC; ++mc)
            if (ch * C::MC + mc < C::MT)
              dmma884(c2[mc][n2][0], c2[mc][n2][1], t1[mc][nt][e], e ? b[n2].y : b[n2].x);
    }
  } else {  // EB = row-major (-1)^{|q|} E~_cd^T of the primitive pair
    const int g = lane >> 2, t = lane & 3;
#pragma unroll
    for (int nt = 0; nt < C::NT1; ++nt)
#pragma unroll
      for (int e = 0; e < 2; ++e) {
        const int qq = 8 * nt + 2 * t + e;
#pragma unroll
        for (int n2 = 0; n2 < C::NT2; ++n2) {
          const int cd = 8 * n2 + g;
          const double b = (qq < C::NHCD && cd < C::NCD) ? __ldg(EB + qq * C::NCD + cd) : 0.0;
#pragma unroll
          for (int mc = 0; mc < C::MC; ++mc)
            if (ch * C::MC + mc < C::MT) dmma884(c2[mc][n2][0], c2[mc][n2][1], t1[mc][nt][e], b);
        }
      }
  }
}

template <int L>
__device__ __forceinline__ void r_regs(double p, double Px, double Py, double Pz, double q, double Qx, double Qy,
                                       double Qz, const double* __restrict__ btab, double (&R)[nH(L)]);

// Batched-R variant of quartet_block for contracted quartets (K_AB K_CD > 1, K_AB <= RB): per batch of
// floor(RB / K_AB) ket primitives, lane c computes the whole R^{(0)} of primitive quartet
// (bra primitive c % K_AB, ket primitive c / K_AB) in registers (Boys + Eq. 5 unrolled, the striped
// layout of PAPER.md:L233-L237) and stores it to row c of the warp's R rows (the SL -> BL hand-off);
// the GEMM1 of a ket primitive then runs over all K_AB rows before its single register-chained GEMM2.
template <class C>
__device__ void quartet_block_rb(const PairView& bra, int b0, int KAB, const PairView& ket, int k0, int k1,
                                 double* __restrict__ Rbuf, double* __restrict__ V, const uint16_t* __restrict__ htab,
                                 const double* __restrict__ btab, int lane) {
  constexpr int RB = C::RB, RS = C::RS, L = C::L;
  constexpr bool ONECHUNK = C::NCHUNK == 1 && 2 * C::MC * (C::NT1 + C::NT2) <= 24;
  const int g = lane >> 2, t = lane & 3;
  if constexpr (!ONECHUNK)
    for (int i = lane; i < C::NAB * C::NCD; i += 32) V[i] = 0.0;
  double c2[C::MC][C::NT2][2];
#pragma unroll
  for (int mc = 0; mc < C::MC; ++mc)
#pragma unroll
    for (int n2 = 0; n2 < C::NT2; ++n2) c2[mc][n2][0] = c2[mc][n2][1] = 0.0;
  const int nkb = RB / KAB;
  for (int kb = k0; kb < k1; kb += nkb) {
    const int nk = min(nkb, k1 - kb);
    if (lane < nk * KAB) {
      const int kl = kb + lane / KAB, ij = b0 + lane % KAB;
      double p, Px, Py, Pz, q, Qx, Qy, Qz;
      load_pdat<true>(bra.pdat, ij, p, Px, Py, Pz);
      load_pdat<true>(ket.pdat, kl, q, Qx, Qy, Qz);
      double Rr[nH(L)];
      r_regs<L>(p, Px, Py, Pz, q, Qx, Qy, Qz, btab, Rr);
      double* row = Rbuf + lane * RS;
#pragma unroll
      for (int h = 0; h < nH(L); ++h) row[h] = Rr[h];
    }
    __syncwarp();
    for (int k = 0; k < nk; ++k) {
      const double* __restrict__ EB = C::FRAGB ? ket.EketD + (size_t)(kb + k) * frag_b_doubles(C::LC, C::LD)
                                                  : ket.Eket + (size_t)(kb + k) * (C::NHCD * C::NCD);
      for (int ch = 0; ch < C::NCHUNK; ++ch) {
        double t1[C::MC][C::NT1][2];
#pragma unroll
        for (int mc = 0; mc < C::MC; ++mc)
#pragma unroll
          for (int nt = 0; nt < C::NT1; ++nt) t1[mc][nt][0] = t1[mc][nt][1] = 0.0;
        for (int il = 0; il < KAB; ++il)
          gemm1_row<C>(t1, ebra_ptr<C>(bra, b0 + il), Rbuf + (k * KAB + il) * RS, htab, ch, lane);
        if constexpr (!ONECHUNK) {
#pragma unroll
          for (int mc = 0; mc < C::MC; ++mc)
#pragma unroll
            for (int n2 = 0; n2 < C::NT2; ++n2) c2[mc][n2][0] = c2[mc][n2][1] = 0.0;
        }
        gemm2_chain<C>(c2, t1, EB, ch, lane);
        if constexpr (!ONECHUNK) {
#pragma unroll
          for (int mc = 0; mc < C::MC; ++mc)
#pragma unroll
            for (int n2 = 0; n2 < C::NT2; ++n2)
#pragma unroll
              for (int i = 0; i < 2; ++i) {
                const int row = 8 * (ch * C::MC + mc) + g, col = 8 * n2 + 2 * t + i;
                if (row < C::NAB && col < C::NCD) V[row * C::NCD + col] += c2[mc][n2][i];
              }
        }
      }
    }
    __syncwarp();  // R rows are overwritten by the next batch
  }
  if constexpr (ONECHUNK) {
#pragma unroll
    for (int mc = 0; mc < C::MC; ++mc)
#pragma unroll
      for (int n2 = 0; n2 < C::NT2; ++n2)
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int row = 8 * mc + g, col = 8 * n2 + 2 * t + i;
          if (row < C::NAB && col < C::NCD) V[row * C::NCD + col] = c2[mc][n2][i];
        }
  }
  __syncwarp();
}

// (ab|cd) block for bra pair P of `bra` and ket pair R of `ket` into V[ab][cd] (warp SMEM).
// m8n8k4 f64 fragments (lane = 4g + t): A[g][t]; B[k=t][n=g]; C[g][2t+i].
// Per ket primitive: R is computed once for up to KR bra primitives into SMEM rows; every row chunk
// (MC m-tiles, bounded by the accumulator register budget) then runs GEMM1 over those rows and the
// register-chained GEMM2, and adds its rows of (ab|cd) into V.
template <class C>
__device__ void quartet_block(const PairView& bra, int P, const PairView& ket, int R, double* __restrict__ Rbuf,
                              double* __restrict__ V, const uint16_t* __restrict__ htab,
                              const uint32_t* __restrict__ rtab, const double* __restrict__ btab, int lane) {
  constexpr int KR = C::KR, NH = C::NH;
  // one row chunk with small accumulators: the GEMM2 accumulators stay in registers across all
  // primitive quartets and V is written once; otherwise each chunk adds its rows into V (SMEM)
  constexpr bool ONECHUNK = C::NCHUNK == 1 && 2 * C::MC * (C::NT1 + C::NT2) <= 24;
  const int g = lane >> 2, t = lane & 3;
  const int b0 = __ldg(bra.poff + P), b1 = __ldg(bra.poff + P + 1);
  const int k0 = __ldg(ket.poff + R), k1 = __ldg(ket.poff + R + 1);
  if constexpr (C::RBATCH) {
    if ((b1 - b0) * (k1 - k0) > 1 && b1 - b0 <= C::RB) {
      quartet_block_rb<C>(bra, b0, b1 - b0, ket, k0, k1, Rbuf, V, htab, btab, lane);
      return;
    }
  }
  if constexpr (!ONECHUNK)
    for (int i = lane; i < C::NAB * C::NCD; i += 32) V[i] = 0.0;
  double c2[C::MC][C::NT2][2];
#pragma unroll
  for (int mc = 0; mc < C::MC; ++mc)
#pragma unroll
    for (int n2 = 0; n2 < C::NT2; ++n2) c2[mc][n2][0] = c2[mc][n2][1] = 0.0;
  for (int kl = k0; kl < k1; ++kl) {
    double q, Qx, Qy, Qz;
    load_pdat(ket.pdat, kl, q, Qx, Qy, Qz);
    const double* __restrict__ EB = C::FRAGB ? ket.EketD + (size_t)kl * frag_b_doubles(C::LC, C::LD)
                                                : ket.Eket + (size_t)kl * (C::NHCD * C::NCD);
    // single row chunk and one R row: stream the bra primitives through it, GEMM2 once per ket primitive
    constexpr bool STREAM = C::NCHUNK == 1 && KR == 1;
    double t1s[C::MC][C::NT1][2];
    if constexpr (STREAM) {
#pragma unroll
      for (int mc = 0; mc < C::MC; ++mc)
#pragma unroll
        for (int nt = 0; nt < C::NT1; ++nt) t1s[mc][nt][0] = t1s[mc][nt][1] = 0.0;
    }
    for (int ig0 = b0; ig0 < b1; ig0 += KR) {
      const int ign = min(KR, b1 - ig0);
      for (int il = 0; il < ign; ++il) {
        double p, Px, Py, Pz;
        load_pdat(bra.pdat, ig0 + il, p, Px, Py, Pz);
        compute_R<C>(p, Px, Py, Pz, q, Qx, Qy, Qz, Rbuf + il * NH, Rbuf + KR * NH, rtab, btab, lane);
      }
      for (int ch = 0; ch < C::NCHUNK; ++ch) {
        double t1[C::MC][C::NT1][2];
#pragma unroll
        for (int mc = 0; mc < C::MC; ++mc)
#pragma unroll
          for (int nt = 0; nt < C::NT1; ++nt) {
            t1[mc][nt][0] = STREAM ? t1s[mc][nt][0] : 0.0;
            t1[mc][nt][1] = STREAM ? t1s[mc][nt][1] : 0.0;
          }
        for (int il = 0; il < ign; ++il)
          gemm1_row<C>(t1, ebra_ptr<C>(bra, ig0 + il), Rbuf + il * NH, htab, ch, lane);
        if constexpr (STREAM) {
          // keep accumulating over the next bra primitives; GEMM2 after the last one
#pragma unroll
          for (int mc = 0; mc < C::MC; ++mc)
#pragma unroll
            for (int nt = 0; nt < C::NT1; ++nt) {
              t1s[mc][nt][0] = t1[mc][nt][0];
              t1s[mc][nt][1] = t1[mc][nt][1];
            }
          if (ig0 + KR < b1) continue;
        }
        if constexpr (!ONECHUNK) {
#pragma unroll
          for (int mc = 0; mc < C::MC; ++mc)
#pragma unroll
            for (int n2 = 0; n2 < C::NT2; ++n2) c2[mc][n2][0] = c2[mc][n2][1] = 0.0;
        }
        gemm2_chain<C>(c2, t1, EB, ch, lane);
        if constexpr (!ONECHUNK) {
#pragma unroll
          for (int mc = 0; mc < C::MC; ++mc)
#pragma unroll
            for (int n2 = 0; n2 < C::NT2; ++n2)
#pragma unroll
              for (int i = 0; i < 2; ++i) {
                const int row = 8 * (ch * C::MC + mc) + g, col = 8 * n2 + 2 * t + i;
                if (row < C::NAB && col < C::NCD) V[row * C::NCD + col] += c2[mc][n2][i];
              }
        }
      }
      __syncwarp();  // R rows are overwritten by the next bra-primitive group
    }
  }
  if constexpr (ONECHUNK) {
#pragma unroll
    for (int mc = 0; mc < C::MC; ++mc)
#pragma unroll
      for (int n2 = 0; n2 < C::NT2; ++n2)
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int row = 8 * mc + g, col = 8 * n2 + 2 * t + i;
          if (row < C::NAB && col < C::NCD) V[row * C::NCD + col] = c2[mc][n2][i];
        }
  }
  __syncwarp();
}

// Orientation of an R x C block of J/K updates in the non-symmetrised accumulators (J = Jacc + Jacc^T,
// K = Kacc + Kacc^T at the end of the build, so element (r, c) may go to (r, c) or (c, r)).  blk_rc maps
// the y-th element of the block to (r, c) so that consecutive y are adjacent in memory; blk_dst is its
// accumulator offset.  FLIP allows the transposed orientation when it gives longer runs (R > C); the
// K blocks never flip: their rows are the task's bra shells, and keeping every update of a task in
// those few rows is what keeps them L2-resident (flipped, the (dp|pp) slab kernel ran 16 % slower).
template <int R, int C, bool FLIP = false>
__device__ __forceinline__ void blk_rc(int y, int& r, int& c) {
  if constexpr (FLIP && R > C) { c = y / R; r = y % R; }
  else { r = y / C; c = y % C; }
}
template <int R, int C, bool FLIP = false>
__device__ __forceinline__ size_t blk_dst(int row, int col, int nbf) {
  if constexpr (FLIP && R > C) return (size_t)col * nbf + row;
  else return (size_t)row * nbf + col;
}

// Digestion of one canonical quartet (north_star J/K; FP64 accumulation).
// With v' = deg * (ab|cd), deg = 1/2 per coincidence (a=b, c=d, ab=cd), the 8 permutations of a
// canonical quartet reduce for symmetric D to the 6 forward updates below; the transposed halves
// are restored by J = Jacc + Jacc^T, K = Kacc + Kacc^T at the end of the build.
// V is the warp-SMEM block V[ab][cd] (row stride NCD).  Steps:
//   1. the six D sub-blocks are staged in warp SMEM (Ds) with coalesced row loads;
//   2. J_ab: row pass (lane = ab), accumulated in SMEM over the kets of a task;
//   3. one column pass (lane = cd = (c,d)) reads every V element ONCE and forms, in registers,
//        K_ac partial  sum_b v D_bd   (per a)      K_ad partial  sum_b v D_bc   (per a)
//        K_bc partial  sum_a v D_ad   (per b)      K_bd partial  sum_a v D_ac   (per b)
//        J_cd          sum_ab v D_ab  (complete per lane)
//      the K partials go to SMEM (Ps) as [a or b][cd];
//   4. K_ac/K_bc sum their partials over d, K_ad/K_bd over c, one FP64 atomic per K element.
template <class C>
struct DigestLayout {
  static constexpr int AB = 0, CD = AB + C::NA * C::NB, AC = CD + C::NC * C::ND, AD = AC + C::NA * C::NC,
                       BC = AD + C::NA * C::ND, BD = BC + C::NB * C::NC, TOT = BD + C::NB * C::ND;
  // partial sums (Ps): [NA][NCD] x 2, [NB][NCD] x 2
  static constexpr int PAC = 0, PAD = PAC + C::NA * C::NCD, PBC = PAD + C::NA * C::NCD, PBD = PBC + C::NB * C::NCD,
                       PTOT = PBD + C::NB * C::NCD;
};

// offset in D of staged element x (D_ab | D_cd | D_ac | D_ad | D_bc | D_bd)
template <class C>
__device__ __forceinline__ size_t d_offset(int x, int oa, int ob, int oc, int od, int nbf) {
  using DL = DigestLayout<C>;
  constexpr int NB = C::NB, NC = C::NC, ND = C::ND;
  int r, c;
  if (x < DL::CD) { r = oa + (x - DL::AB) / NB; c = ob + (x - DL::AB) % NB; }
  else if (x < DL::AC) { r = oc + (x - DL::CD) / ND; c = od + (x - DL::CD) % ND; }
  else if (x < DL::AD) { r = oa + (x - DL::AC) / NC; c = oc + (x - DL::AC) % NC; }
  else if (x < DL::BC) { r = oa + (x - DL::AD) / ND; c = od + (x - DL::AD) % ND; }
  else if (x < DL::BD) { r = ob + (x - DL::BC) / NC; c = oc + (x - DL::BC) % NC; }
  else { r = ob + (x - DL::BD) / ND; c = od + (x - DL::BD) % ND; }
  return (size_t)r * nbf + c;
}

// D sub-blocks of one quartet copied to warp SMEM asynchronously (cp.async), issued before the
// quartet's ERI work and waited for before its digestion: the L2 latency of the scattered D reads is
// hidden behind the ERI evaluation
template <class C>
__device__ __forceinline__ void d_prefetch(double* __restrict__ Ds, const double* __restrict__ D, int oa, int ob,
                                           int oc, int od, int nbf, int lane) {
  for (int x = lane; x < DigestLayout<C>::TOT; x += 32) cp_async8(Ds + x, D + d_offset<C>(x, oa, ob, oc, od, nbf));
  cp_async_commit();
}

template <class C, bool STAGE = true>
__device__ void digest(const double* __restrict__ V, double deg, int oa, int ob, int oc, int od,
                       const double* __restrict__ D, int nbf, double* __restrict__ J, double* __restrict__ K,
                       double* __restrict__ jab, double* __restrict__ Ds, double* __restrict__ Ps, int lane) {
  using DL = DigestLayout<C>;
  constexpr int NA = C::NA, NB = C::NB, NC = C::NC, ND = C::ND, NCD = C::NCD;
  // 1. stage D_ab, D_cd, D_ac, D_ad, D_bc, D_bd (unless the caller prefetched them: d_prefetch)
  if constexpr (STAGE) {
    for (int x = lane; x < DL::TOT; x += 32) Ds[x] = __ldg(D + d_offset<C>(x, oa, ob, oc, od, nbf));
  } else {
    cp_async_wait_all();
  }
  __syncwarp();
  const double* Dab = Ds + DL::AB;
  const double* Dcd = Ds + DL::CD;
  // 2. J_ab (row pass; odd row stride NCD keeps it bank-conflict free)
  for (int ab = lane; ab < C::NAB; ab += 32) {
    double s0 = 0.0, s1 = 0.0;
    int cd = 0;
    for (; cd + 1 < NCD; cd += 2) {
      s0 = fma(V[ab * NCD + cd], Dcd[cd], s0);
      s1 = fma(V[ab * NCD + cd + 1], Dcd[cd + 1], s1);
    }
    if (cd < NCD) s0 = fma(V[ab * NCD + cd], Dcd[cd], s0);
    jab[ab] = fma(2.0 * deg, s0 + s1, jab[ab]);
  }
  // 3. column pass
  for (int cd = lane; cd < NCD; cd += 32) {
    const int c = cd / ND, d = cd % ND;
    double dbd[NB], dbc[NB], kbc[NB], kbd[NB];
#pragma unroll
    for (int b = 0; b < NB; ++b) {
      dbd[b] = Ds[DL::BD + b * ND + d];
      dbc[b] = Ds[DL::BC + b * NC + c];
      kbc[b] = 0.0;
      kbd[b] = 0.0;
    }
    double jcd0 = 0.0, jcd1 = 0.0;
#pragma unroll
    for (int a = 0; a < NA; ++a) {
      const double dad = Ds[DL::AD + a * ND + d], dac = Ds[DL::AC + a * NC + c];
      double kac = 0.0, kad = 0.0;
#pragma unroll
      for (int b = 0; b < NB; ++b) {
        const double v = V[(a * NB + b) * NCD + cd];
        kac = fma(v, dbd[b], kac);
        kad = fma(v, dbc[b], kad);
        kbc[b] = fma(v, dad, kbc[b]);
        kbd[b] = fma(v, dac, kbd[b]);
        if (b & 1) jcd1 = fma(v, Dab[a * NB + b], jcd1); else jcd0 = fma(v, Dab[a * NB + b], jcd0);
      }
      Ps[DL::PAC + a * NCD + cd] = kac;
      Ps[DL::PAD + a * NCD + cd] = kad;
    }
#pragma unroll
    for (int b = 0; b < NB; ++b) {
      Ps[DL::PBC + b * NCD + cd] = kbc[b];
      Ps[DL::PBD + b * NCD + cd] = kbd[b];
    }
    atomicAdd(J + (size_t)(oc + c) * nbf + od + d, 2.0 * deg * (jcd0 + jcd1));
  }
  __syncwarp();
  // 4. K_ac[a][c] = sum_d P_ac[a][c,d] | K_ad[a][d] = sum_c P_ad[a][c,d] |
  //    K_bc[b][c] = sum_d P_bc[b][c,d] | K_bd[b][d] = sum_c P_bd[b][c,d]
  //    Consecutive lanes take adjacent columns of a bra row, so one RED instruction covers runs of NC
  //    or ND adjacent doubles (the L2 atomic units work per 32-byte sector: measured 1.65e11 sectors/s,
  //    4.2e11 doubles/s with 4 doubles per sector, tools/atomics_bench.cu)
  constexpr int N1 = NA * NC, N2 = N1 + NA * ND, N3 = N2 + NB * NC, N4 = N3 + NB * ND;
  constexpr int NMX = NC > ND ? NC : ND;
  for (int x = lane; x < N4; x += 32) {
    int base, stride, cnt;
    size_t dst;
    if (x < N1) {
      int i, k;
      blk_rc<NA, NC>(x, i, k);
      base = DL::PAC + i * NCD + k * ND; stride = 1; cnt = ND; dst = blk_dst<NA, NC>(oa + i, oc + k, nbf);
    } else if (x < N2) {
      int i, l;
      blk_rc<NA, ND>(x - N1, i, l);
      base = DL::PAD + i * NCD + l; stride = ND; cnt = NC; dst = blk_dst<NA, ND>(oa + i, od + l, nbf);
    } else if (x < N3) {
      int j, k;
      blk_rc<NB, NC>(x - N2, j, k);
      base = DL::PBC + j * NCD + k * ND; stride = 1; cnt = ND; dst = blk_dst<NB, NC>(ob + j, oc + k, nbf);
    } else {
      int j, l;
      blk_rc<NB, ND>(x - N3, j, l);
      base = DL::PBD + j * NCD + l; stride = ND; cnt = NC; dst = blk_dst<NB, ND>(ob + j, od + l, nbf);
    }
    double s = 0.0;
#pragma unroll
    for (int k = 0; k < NMX; ++k)
      if (k < cnt) s += Ps[base + k * stride];
    atomicAdd(K + dst, deg * s);
  }
  __syncwarp();
}

}  // namespace mako
