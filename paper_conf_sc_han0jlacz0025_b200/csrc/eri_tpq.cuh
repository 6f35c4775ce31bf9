// eri_tpq.cuh -- lane-per-ket register kernel for the low angular-momentum classes.
//
// The paper's "striped layout" (S3.1.2: one thread per shell quartet, each
// parameter strided by the batch) taken to its end for classes whose whole MMD state fits in
// registers: a warp owns one bra pair and 32 consecutive kets of its Q-sorted prefix; lane i
// evaluates quartet (bra | ket_i) completely in registers:
//   Boys F_m (a4) -> R^{(0)}_{tuv} by Eq. 5 fully unrolled at compile time (a5) ->
//   W[p][cd] = sum_q R_{p+q} (-1)^{|q|} E~_cd[q][cd]  then  V[ab][cd] += E~_ab[ab][p] W[p][cd]
//   (Eq. 7 with the cheaper contraction order for a low-l ket; the bra E~ is warp-uniform) ->
//   digestion (a9): J_ab by warp reduction, J_cd / K blocks by FP64 atomics from each lane.
#pragma once

#include <utility>

#include "eri_core.cuh"

namespace mako {

// compile-time Hermite decode (degree-major, t desc, u desc)
MK_HD constexpr int hd_k(int e) { int k = 0; while (nH(k) <= e) ++k; return k; }
MK_HD constexpr int hd_s(int e) {
  int r = e - nH(hd_k(e) - 1), s = 0;
  while ((s + 1) * (s + 2) / 2 <= r) ++s;
  return s;
}
MK_HD constexpr int hd_v(int e) { return e - nH(hd_k(e) - 1) - hd_s(e) * (hd_s(e) + 1) / 2; }
MK_HD constexpr int hd_u(int e) { return hd_s(e) - hd_v(e); }
MK_HD constexpr int hd_t(int e) { return hd_k(e) - hd_s(e); }
MK_HD constexpr int r_dir(int e) { return hd_t(e) > 0 ? 0 : (hd_u(e) > 0 ? 1 : 2); }
MK_HD constexpr int r_n(int e) { return r_dir(e) == 0 ? hd_t(e) : (r_dir(e) == 1 ? hd_u(e) : hd_v(e)); }
MK_HD constexpr int r_src(int e, int m) {  // index of e - m * 1_dir
  return r_dir(e) == 0 ? hidx(hd_t(e) - m, hd_u(e), hd_v(e))
                       : (r_dir(e) == 1 ? hidx(hd_t(e), hd_u(e) - m, hd_v(e)) : hidx(hd_t(e), hd_u(e), hd_v(e) - m));
}
MK_HD constexpr int h_sum(int p, int q) {
  return hidx(hd_t(p) + hd_t(q), hd_u(p) + hd_u(q), hd_v(p) + hd_v(q));
}

template <int B, int E, class F>
__device__ __forceinline__ void static_for(F&& f) {
  if constexpr (B < E) {
    f(std::integral_constant<int, B>{});
    static_for<B + 1, E>(f);
  }
}

// NH x NC doubles (contiguous, 16 B aligned when NH*NC is even) into a register matrix
template <int NH, int NC>
__device__ __forceinline__ void load_mat(const double* __restrict__ src, double (&M)[NH][NC]) {
  if constexpr ((NH * NC) % 4 == 0) {  // 32 B aligned rows of the E~ array: 256-bit loads
    static_for<0, NH * NC / 4>([&](auto ic) {
      constexpr int i = decltype(ic)::value;
      double w0, w1, w2, w3;
      ldg256(src + 4 * i, w0, w1, w2, w3);
      M[(4 * i) / NC][(4 * i) % NC] = w0;
      M[(4 * i + 1) / NC][(4 * i + 1) % NC] = w1;
      M[(4 * i + 2) / NC][(4 * i + 2) % NC] = w2;
      M[(4 * i + 3) / NC][(4 * i + 3) % NC] = w3;
    });
  } else if constexpr ((NH * NC) % 2 == 0) {
    const double2* v = reinterpret_cast<const double2*>(src);
    static_for<0, NH * NC / 2>([&](auto ic) {
      constexpr int i = decltype(ic)::value;
      const double2 w = __ldg(v + i);
      M[(2 * i) / NC][(2 * i) % NC] = w.x;
      M[(2 * i + 1) / NC][(2 * i + 1) % NC] = w.y;
    });
  } else {
#pragma unroll
    for (int h = 0; h < NH; ++h)
#pragma unroll
      for (int j = 0; j < NC; ++j) M[h][j] = __ldg(src + h * NC + j);
  }
}

// one level of the in-place R recursion: entries E, E-1, ..., 1 (descending = degree-descending,
// so every source of level n+1 is still unmodified when read)
template <int E>
__device__ __forceinline__ void r_level(double* R, double X, double Y, double Z) {
  if constexpr (E >= 1) {
    constexpr int dir = r_dir(E), n = r_n(E), s1 = r_src(E, 1);
    const double x = dir == 0 ? X : (dir == 1 ? Y : Z);
    if constexpr (n >= 2) {
      constexpr int s2 = r_src(E, 2);
      R[E] = fma((double)(n - 1), R[s2], x * R[s1]);
    } else {
      R[E] = x * R[s1];
    }
    r_level<E - 1>(R, X, Y, Z);
  }
}

template <int L, int N>
__device__ __forceinline__ void r_levels(double* R, const double* F, double X, double Y, double Z) {
  if constexpr (N >= 0) {
    r_level<nH(L - N) - 1>(R, X, Y, Z);
    R[0] = F[N];
    r_levels<L, N - 1>(R, F, X, Y, Z);
  }
}

// Boys + R^{(0)} into registers (R[nH(L)]), seeds scaled by 2 pi^{5/2}/sqrt(p+q) (-2 rho)^n
template <int L>
__device__ __forceinline__ void r_regs(double p, double Px, double Py, double Pz, double q, double Qx, double Qy,
                                       double Qz, const double* __restrict__ btab, double (&R)[nH(L)]) {
  const double pq = p + q, ri = rsqrt_fast(pq), rho = p * q * ri * ri;
  const double X = Px - Qx, Y = Py - Qy, Z = Pz - Qz;
  double F[L + 1];
  boys_eval<L, true>(rho * (X * X + Y * Y + Z * Z), btab, F);
  double s = TWO_PI_52 * ri;
  const double m2r = -2.0 * rho;
#pragma unroll
  for (int n = 0; n <= L; ++n) {
    F[n] *= s;
    s *= m2r;
  }
  R[0] = F[L];
  r_levels<L, L - 1>(R, F, X, Y, Z);
}

// W-accumulation variant fits in registers (R + V + W + ket E~, doubles)?
template <class C>
constexpr bool tpq_wacc() {
  return nH(C::L) + C::NAB * C::NCD + C::NHAB * C::NCD + C::NHCD * C::NCD <= 110;
}

// One grab of the persistent task loop: lane 0 takes TASK_GRAB local tasks from the class counter;
// returns false when the shard's tasks are exhausted, else the global task range [tg0, tg1) (never
// crosses a shard chunk: chunk sizes are multiples of TASK_GRAB and grabs start at multiples of it).
__device__ __forceinline__ bool grab_tasks(const JKArgs& a, int lane, long long& tg0, long long& tg1) {
  unsigned long long grab = 0;
  if (lane == 0) grab = atomicAdd(a.counter, (unsigned long long)TASK_GRAB);
  grab = __shfl_sync(0xffffffffu, grab, 0);
  const long long l0 = (long long)grab;
  if (l0 >= a.ntask_local) return false;
  tg0 = a.nshards == 1 ? l0 : shard_task(l0, a.shard, a.nshards, a.chunk);
  tg1 = min(tg0 + TASK_GRAB, a.ntask);
  return true;
}

// density-weighted screening of quartet (sa sb|sc sd) with Schwarz product qq (reading R17)
template <bool DW>
__device__ __forceinline__ bool dw_keep(const JKArgs& a, double qq, int sa, int sb, int sc, int sd) {
  if constexpr (!DW) return true;
  const float* __restrict__ t = a.dsh;
  const size_t n = (size_t)a.nshell;
  const float m = fmaxf(fmaxf(__ldg(t + sa * n + sb), __ldg(t + sc * n + sd)),
                        fmaxf(fmaxf(__ldg(t + sa * n + sc), __ldg(t + sa * n + sd)),
                              fmaxf(__ldg(t + sb * n + sc), __ldg(t + sb * n + sd))));
  return qq * (double)m * (1.0 + 1e-6) >= a.dw_thresh;  // (float rounding of the block maxima)
}

// entry (non-empty bra pair x ket K-group) holding task `task`: sampled start + short forward scan
__device__ __forceinline__ int find_entry(const JKArgs& a, long long task) {
  int U = __ldg(a.usamp + (task >> TASK_SAMPLE_SHIFT));
  while (__ldg(a.task_off + U + 1) <= task) ++U;
  return U;
}

// K-row strip of a bra unit in shared memory (strip digestion, S6): rows 0..NA-1 hold
// K[oa + i][*], rows NA..NA+NB-1 hold K[ob + j][*], full nbf columns; J_ab partial sums behind them;
// a bitmap of the ket shells whose columns were touched.  Flushed to global J/K once per bra unit.
struct Strip {
  double* K;          // [(NA + NB) * nbf]
  double* Jab;        // [NAB]
  unsigned* touched;  // [(nshell + 31) / 32]
};

// shared-memory double add (sm_100a has no native f64 shared atomic: CAS loop, rarely contended here)
__device__ __forceinline__ void sh_add(double* p, double v) { atomicAdd(p, v); }

// Sector-grouped digestion of one R x C block per lane (lane = ket) of the lane-per-ket kernel: the
// lanes' block values go through warp shared memory so that each RED instruction covers, for ~32/run
// kets, a run of adjacent doubles (blk_rc / blk_dst in eri_core.cuh; K blocks stay in the bra rows):
// the L2 atomic units are bound per 32-byte sector, not per double (1.65e11 sectors/s measured,
// tools/atomics_bench.cu), and the direct per-lane atomics hit one sector per double.  Used for p kets
// (runs of 3 adjacent columns); for s kets every run is one double.
#ifndef MAKO_TPQ_STAGE
#define MAKO_TPQ_STAGE 0  // measured: 11.37 s/build without, 11.51 s with (the SMEM round trip costs more)
#endif
template <int R, int CC, bool FLIP, class F>
__device__ __forceinline__ void staged_red(double* __restrict__ out, double* __restrict__ stage, int lane, bool active,
                                           int orow, int ocol, int nbf, F&& val) {
  constexpr int E = R * CC;
#pragma unroll
  for (int y = 0; y < E; ++y) {
    int r, c;
    blk_rc<R, CC, FLIP>(y, r, c);
    stage[lane * E + y] = active ? val(r, c) : 0.0;
  }
  __syncwarp();
#pragma unroll
  for (int it = 0; it < E; ++it) {
    const int idx = it * 32 + lane, ket = idx / E, y = idx % E;
    const int orw = __shfl_sync(0xffffffffu, orow, ket), ocl = __shfl_sync(0xffffffffu, ocol, ket);
    const double v = stage[idx];
    int r, c;
    blk_rc<R, CC, FLIP>(y, r, c);
    if (v != 0.0) atomicAdd(out + blk_dst<R, CC, FLIP>(orw + r, ocl + c, nbf), v);
  }
  __syncwarp();
}
template <class C>
__host__ __device__ constexpr int tpq_stage_doubles() {
  constexpr int a = C::NA * C::NC, b = C::NA * C::ND, c = C::NB * C::NC, d = C::NB * C::ND, e = C::NC * C::ND;
  constexpr int m1 = a > b ? a : b, m2 = c > d ? c : d, m3 = m1 > m2 ? m1 : m2;
  return 32 * (m3 > e ? m3 : e);
}

// One lane-per-ket task: bra pair P, kets [r0, r1) (<= 32, lane i takes ket r0 + i).  Boys, R, the
// ket-first contraction and digestion all in registers.  STRIP: the K_ac/K_ad/K_bc/K_bd updates and
// J_ab go to the CTA's shared K-row strip of bra P instead of global FP64 atomics (J_cd stays global).
template <int X, int Y, bool DW, bool STRIP>
__device__ __forceinline__ void tpq_task(const JKArgs& a, int P, int r0, int r1, int lane, const Strip& st,
                                         double* __restrict__ stage = nullptr) {
  using C = ClsXY<X, Y>;
  constexpr int NAB = C::NAB, NCD = C::NCD, NHAB = C::NHAB, NHCD = C::NHCD, L = C::L;
  constexpr int NA = C::NA, NB = C::NB, NC = C::NC, ND = C::ND;
  constexpr bool WACC = tpq_wacc<C>();
    const int R = r0 + lane;
    const double QP = __ldg(a.bra.Q + P);
    const double QQ = QP * __ldg(a.ket.Q + min(R, r1 - 1));
    const int sa = __ldg(a.bra.shA + P), sb = __ldg(a.bra.shB + P);
    const bool active = R < r1 && QQ >= a.thresh &&
                        dw_keep<DW>(a, QQ, sa, sb, __ldg(a.ket.shA + min(R, r1 - 1)), __ldg(a.ket.shB + min(R, r1 - 1)));
    const int oa = __ldg(a.ao + sa), ob = __ldg(a.ao + sb);
    const int b0 = __ldg(a.bra.poff + P), b1 = __ldg(a.bra.poff + P + 1);
    double V[NAB][NCD];
#pragma unroll
    for (int i = 0; i < NAB; ++i)
#pragma unroll
      for (int j = 0; j < NCD; ++j) V[i][j] = 0.0;
    int sc = 0, sd = 0;
    if (active) {
      sc = __ldg(a.ket.shA + R);
      sd = __ldg(a.ket.shB + R);
    }
    if (active) {
      const int k0 = __ldg(a.ket.poff + R), k1 = __ldg(a.ket.poff + R + 1);
      if constexpr (WACC) {
        // bra primitive outer: W[p][cd] = sum_kl sum_q R_{p+q} E~_cd[q][cd], then V += E~_ab W
        for (int ij = b0; ij < b1; ++ij) {
          double p, Px, Py, Pz;
        load_pdat(a.bra.pdat, ij, p, Px, Py, Pz);
          double W[NHAB][NCD];
#pragma unroll
          for (int h = 0; h < NHAB; ++h)
#pragma unroll
            for (int j = 0; j < NCD; ++j) W[h][j] = 0.0;
          for (int kl = k0; kl < k1; ++kl) {
            double q, Qx, Qy, Qz;
        load_pdat<true>(a.ket.pdat, kl, q, Qx, Qy, Qz);
            double Ek[NHCD][NCD];
            const double* __restrict__ ek = a.ket.Eket + (size_t)kl * (NHCD * NCD);
            load_mat<NHCD, NCD>(ek, Ek);
            double Rr[nH(L)];
            r_regs<L>(p, Px, Py, Pz, q, Qx, Qy, Qz, a.boys, Rr);
            static_for<0, NHAB>([&](auto pc) {
              constexpr int pp = decltype(pc)::value;
              static_for<0, NHCD>([&](auto qc) {
                constexpr int qq = decltype(qc)::value;
                constexpr int hs = h_sum(pp, qq);
#pragma unroll
                for (int j = 0; j < NCD; ++j) W[pp][j] = fma(Rr[hs], Ek[qq][j], W[pp][j]);
              });
            });
          }
          const double* __restrict__ eb = a.bra.Ebra + (size_t)ij * (NAB * NHAB);
#pragma unroll
          for (int i = 0; i < NAB; ++i)
#pragma unroll
            for (int h = 0; h < NHAB; ++h) {
              const double e = __ldg(eb + i * NHAB + h);
#pragma unroll
              for (int j = 0; j < NCD; ++j) V[i][j] = fma(e, W[h][j], V[i][j]);
            }
        }
      } else {
      for (int kl = k0; kl < k1; ++kl) {
        double q, Qx, Qy, Qz;
        load_pdat<true>(a.ket.pdat, kl, q, Qx, Qy, Qz);
        // signed ket E~^T [q][cd]
        double Ek[NHCD][NCD];
        const double* __restrict__ ek = a.ket.Eket + (size_t)kl * (NHCD * NCD);
        load_mat<NHCD, NCD>(ek, Ek);
        for (int ij = b0; ij < b1; ++ij) {
          double p, Px, Py, Pz;
        load_pdat(a.bra.pdat, ij, p, Px, Py, Pz);
          double Rr[nH(L)];
          r_regs<L>(p, Px, Py, Pz, q, Qx, Qy, Qz, a.boys, Rr);
          const double* __restrict__ eb = a.bra.Ebra + (size_t)ij * (NAB * NHAB);
          static_for<0, NHAB>([&](auto pc) {
            constexpr int pp = decltype(pc)::value;
            double W[NCD];
#pragma unroll
            for (int j = 0; j < NCD; ++j) W[j] = 0.0;
            static_for<0, NHCD>([&](auto qc) {
              constexpr int qq = decltype(qc)::value;
              constexpr int hs = h_sum(pp, qq);
#pragma unroll
              for (int j = 0; j < NCD; ++j) W[j] = fma(Rr[hs], Ek[qq][j], W[j]);
            });
#pragma unroll
            for (int i = 0; i < NAB; ++i) {
              const double e = __ldg(eb + i * NHAB + pp);
#pragma unroll
              for (int j = 0; j < NCD; ++j) V[i][j] = fma(e, W[j], V[i][j]);
            }
          });
        }
      }
      }
    }
    // ---- digestion (a9) ----
    double deg = 1.0;
    if (sa == sb) deg *= 0.5;
    if (sc == sd) deg *= 0.5;
    if (a.same_bucket && P == R) deg *= 0.5;
    if (!active) deg = 0.0;
    const size_t n = (size_t)a.nbf;
    const int oc = active ? __ldg(a.ao + sc) : 0, od = active ? __ldg(a.ao + sd) : 0;
    const double* __restrict__ Dm = a.D;
    // J_ab: per-lane deg-weighted partial, warp reduction over the 32 kets, one atomic per element
#pragma unroll
    for (int i = 0; i < NAB; ++i) {
      double s = 0.0;
      if (active) {
#pragma unroll
        for (int kl = 0; kl < NCD; ++kl) s = fma(V[i][kl], __ldg(Dm + (oc + kl / ND) * n + od + kl % ND), s);
      }
      s *= deg;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
      if (lane == 0) {
        if constexpr (STRIP) sh_add(st.Jab + i, 2.0 * s);
        else atomicAdd(a.J + (oa + i / NB) * n + ob + i % NB, 2.0 * s);
      }
    }
    if constexpr (!STRIP && MAKO_TPQ_STAGE && NC > 1) {
      const double* __restrict__ Db = Dm;
      // J_cd ; K_ac += v D_bd ; K_ad += v D_bc ; K_bc += v D_ad ; K_bd += v D_ac (deg = 0 on idle lanes)
      staged_red<NC, ND, true>(a.J, stage, lane, active, oc, od, a.nbf, [&](int k, int l) {
        double s = 0.0;
#pragma unroll
        for (int ij = 0; ij < NAB; ++ij) s = fma(V[ij][k * ND + l], __ldg(Db + (oa + ij / NB) * n + ob + ij % NB), s);
        return 2.0 * deg * s;
      });
      staged_red<NA, NC, false>(a.K, stage, lane, active, oa, oc, a.nbf, [&](int i, int k) {
        double s = 0.0;
#pragma unroll
        for (int j = 0; j < NB; ++j)
#pragma unroll
          for (int l = 0; l < ND; ++l) s = fma(V[i * NB + j][k * ND + l], __ldg(Db + (ob + j) * n + od + l), s);
        return deg * s;
      });
      staged_red<NA, ND, false>(a.K, stage, lane, active, oa, od, a.nbf, [&](int i, int l) {
        double s = 0.0;
#pragma unroll
        for (int j = 0; j < NB; ++j)
#pragma unroll
          for (int k = 0; k < NC; ++k) s = fma(V[i * NB + j][k * ND + l], __ldg(Db + (ob + j) * n + oc + k), s);
        return deg * s;
      });
      staged_red<NB, NC, false>(a.K, stage, lane, active, ob, oc, a.nbf, [&](int j, int k) {
        double s = 0.0;
#pragma unroll
        for (int i = 0; i < NA; ++i)
#pragma unroll
          for (int l = 0; l < ND; ++l) s = fma(V[i * NB + j][k * ND + l], __ldg(Db + (oa + i) * n + od + l), s);
        return deg * s;
      });
      staged_red<NB, ND, false>(a.K, stage, lane, active, ob, od, a.nbf, [&](int j, int l) {
        double s = 0.0;
#pragma unroll
        for (int i = 0; i < NA; ++i)
#pragma unroll
          for (int k = 0; k < NC; ++k) s = fma(V[i * NB + j][k * ND + l], __ldg(Db + (oa + i) * n + oc + k), s);
        return deg * s;
      });
      return;
    }
    if (!active) return;
    // J_cd
#pragma unroll
    for (int k = 0; k < NC; ++k)
#pragma unroll
      for (int l = 0; l < ND; ++l) {
        double s = 0.0;
#pragma unroll
        for (int ij = 0; ij < NAB; ++ij) s = fma(V[ij][k * ND + l], __ldg(Dm + (oa + ij / NB) * n + ob + ij % NB), s);
        atomicAdd(a.J + (oc + k) * n + od + l, 2.0 * deg * s);
      }
    if constexpr (STRIP) {
      atomicOr(st.touched + (sc >> 5), 1u << (sc & 31));
      atomicOr(st.touched + (sd >> 5), 1u << (sd & 31));
    }
    // K_ac += v D_bd ; K_ad += v D_bc ; K_bc += v D_ad ; K_bd += v D_ac
    // (strip: row i of shell a is strip row i, row j of shell b is strip row NA + j, column = AO index)
#pragma unroll
    for (int i = 0; i < NA; ++i)
#pragma unroll
      for (int k = 0; k < NC; ++k) {
        double s = 0.0;
#pragma unroll
        for (int j = 0; j < NB; ++j)
#pragma unroll
          for (int l = 0; l < ND; ++l) s = fma(V[i * NB + j][k * ND + l], __ldg(Dm + (ob + j) * n + od + l), s);
        if constexpr (STRIP) sh_add(st.K + i * n + oc + k, deg * s);
        else atomicAdd(a.K + (oa + i) * n + oc + k, deg * s);
      }
#pragma unroll
    for (int i = 0; i < NA; ++i)
#pragma unroll
      for (int l = 0; l < ND; ++l) {
        double s = 0.0;
#pragma unroll
        for (int j = 0; j < NB; ++j)
#pragma unroll
          for (int k = 0; k < NC; ++k) s = fma(V[i * NB + j][k * ND + l], __ldg(Dm + (ob + j) * n + oc + k), s);
        if constexpr (STRIP) sh_add(st.K + i * n + od + l, deg * s);
        else atomicAdd(a.K + (oa + i) * n + od + l, deg * s);
      }
#pragma unroll
    for (int j = 0; j < NB; ++j)
#pragma unroll
      for (int k = 0; k < NC; ++k) {
        double s = 0.0;
#pragma unroll
        for (int i = 0; i < NA; ++i)
#pragma unroll
          for (int l = 0; l < ND; ++l) s = fma(V[i * NB + j][k * ND + l], __ldg(Dm + (oa + i) * n + od + l), s);
        if constexpr (STRIP) sh_add(st.K + (NA + j) * n + oc + k, deg * s);
        else atomicAdd(a.K + (ob + j) * n + oc + k, deg * s);
      }
#pragma unroll
    for (int j = 0; j < NB; ++j)
#pragma unroll
      for (int l = 0; l < ND; ++l) {
        double s = 0.0;
#pragma unroll
        for (int i = 0; i < NA; ++i)
#pragma unroll
          for (int k = 0; k < NC; ++k) s = fma(V[i * NB + j][k * ND + l], __ldg(Dm + (oa + i) * n + oc + k), s);
        if constexpr (STRIP) sh_add(st.K + (NA + j) * n + od + l, deg * s);
        else atomicAdd(a.K + (ob + j) * n + od + l, deg * s);
      }
}

// Persistent lane-per-ket kernel (JKArgs.KT must be 32).  The classes of MAKO_TPQ_CAP3 / MAKO_TPQ_CAP4 are
// compiled for at least 3 / 4 resident CTAs per SM (register caps 168 / 128; measured per class), the
// others without a cap.
#ifndef MAKO_TPQ_CAP3
#define MAKO_TPQ_CAP3 201, 301, 601  // (pp|ps) (ds|ps) (fs|ps): 2 -> 3 CTAs/SM, 380 -> 375, 407 -> 385, 260 -> 241 ms
#endif
#ifndef MAKO_TPQ_CAP4
#define MAKO_TPQ_CAP4 9999
#endif
constexpr int kTpqCap3[] = {MAKO_TPQ_CAP3};
constexpr int kTpqCap4[] = {MAKO_TPQ_CAP4};
template <int X, int Y>
constexpr int tpq_minb() {
  return in_list(kTpqCap4, X * 100 + Y) ? 4 : (in_list(kTpqCap3, X * 100 + Y) ? 3 : 1);
}
template <int X, int Y, bool DW>
__device__ __forceinline__ void tpq_body(const JKArgs& a);
template <int X, int Y, bool DW = false>
__global__ void __launch_bounds__(128) tpq_kernel_free(JKArgs a) { tpq_body<X, Y, DW>(a); }
template <int X, int Y, bool DW = false>
__global__ void __launch_bounds__(128, 3) tpq_kernel_cap3(JKArgs a) { tpq_body<X, Y, DW>(a); }
template <int X, int Y, bool DW = false>
__global__ void __launch_bounds__(128, 4) tpq_kernel_cap4(JKArgs a) { tpq_body<X, Y, DW>(a); }
template <int X, int Y, bool DW = false>
constexpr auto tpq_jk_kernel_ptr() {
  if constexpr (tpq_minb<X, Y>() == 4) return &tpq_kernel_cap4<X, Y, DW>;
  else if constexpr (tpq_minb<X, Y>() == 3) return &tpq_kernel_cap3<X, Y, DW>;
  else return &tpq_kernel_free<X, Y, DW>;
}
template <int X, int Y, bool DW>
__device__ __forceinline__ void tpq_body(const JKArgs& a) {
  const int lane = threadIdx.x & 31;
  __shared__ double stage_all[MAKO_TPQ_STAGE ? 4 * tpq_stage_doubles<ClsXY<X, Y>>() : 1];
  double* stage = stage_all + (MAKO_TPQ_STAGE ? (threadIdx.x >> 5) * tpq_stage_doubles<ClsXY<X, Y>>() : 0);
  for (;;) {
  long long tg0, tg1;
  if (!grab_tasks(a, lane, tg0, tg1)) break;
  int U = find_entry(a, tg0);
  for (long long task = tg0; task < tg1; ++task) {
    while (__ldg(a.task_off + U + 1) <= task) ++U;
    const int P = __ldg(a.ent_P + U);
    const int r0 = __ldg(a.kbeg + U) + (int)(task - __ldg(a.task_off + U)) * 32;
    const int r1 = min(r0 + 32, __ldg(a.kend + U));
    tpq_task<X, Y, DW, false>(a, P, r0, r1, lane, Strip{}, stage);
  }
  }
}

// Strip-digestion variant (S6, "K-row strips"): a CTA takes a whole bra unit (every task of
// one bra pair P, all ket K-groups) from the class's unit counter; its warps share the unit's tasks and
// accumulate K rows of shells a and b (all nbf columns) and J_ab in shared memory; the touched ket-shell
// columns are flushed to global memory with one FP64 atomic per element once per unit.  Per quartet
// the global atomics drop from NCD + (NA+NB)(NC+ND) to NCD (J_cd).  Used when the strip fits in shared
// memory ((NA+NB) nbf doubles); a unit's tasks outside this launch's shard are skipped.
constexpr int TPQ_STRIP_WARPS = 8;
template <int X, int Y>
__host__ __device__ constexpr size_t tpq_strip_smem(int nbf, int nshell) {
  using C = ClsXY<X, Y>;
  return sizeof(double) * ((size_t)(C::NA + C::NB) * nbf + C::NAB) + sizeof(unsigned) * (size_t)((nshell + 31) / 32 + 1);
}
template <int X, int Y, bool DW = false>
__global__ void __launch_bounds__(32 * TPQ_STRIP_WARPS) tpq_strip_kernel(JKArgs a) {
  using C = ClsXY<X, Y>;
  constexpr int NA = C::NA, NB = C::NB, NAB = C::NAB;
  extern __shared__ __align__(16) double strip_smem[];
  __shared__ int s_unit;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nbf = a.nbf, nw = (a.nshell + 31) / 32;
  Strip st;
  st.K = strip_smem;
  st.Jab = strip_smem + (size_t)(NA + NB) * nbf;
  st.touched = reinterpret_cast<unsigned*>(st.Jab + NAB);
  for (int i = threadIdx.x; i < (NA + NB) * nbf + NAB; i += blockDim.x) strip_smem[i] = 0.0;
  for (int i = threadIdx.x; i < nw; i += blockDim.x) st.touched[i] = 0u;
  __syncthreads();
  for (;;) {
    if (threadIdx.x == 0) s_unit = (int)atomicAdd(a.counter, 1ull);
    __syncthreads();
    const int u = s_unit;
    if (u >= a.nunit) break;
    const long long t0 = __ldg(a.unit_off + u), t1 = __ldg(a.unit_off + u + 1);
    const int P = __ldg(a.unit_P + u);
    // the unit's tasks (this shard's part), round-robin over the warps
    int U = -1;
    for (long long task = t0 + warp; task < t1; task += TPQ_STRIP_WARPS) {
      if (a.nshards > 1 && (task / a.chunk) % a.nshards != a.shard) continue;
      if (U < 0) U = find_entry(a, task);
      while (__ldg(a.task_off + U + 1) <= task) ++U;
      const int r0 = __ldg(a.kbeg + U) + (int)(task - __ldg(a.task_off + U)) * 32;
      const int r1 = min(r0 + 32, __ldg(a.kend + U));
      tpq_task<X, Y, DW, true>(a, P, r0, r1, lane, st);
    }
    __syncthreads();
    // flush: J_ab, then the touched columns of the K rows of a and b (zeroing them for the next unit)
    const int sa = __ldg(a.bra.shA + P), sb = __ldg(a.bra.shB + P);
    const int oa = __ldg(a.ao + sa), ob = __ldg(a.ao + sb);
    for (int i = threadIdx.x; i < NAB; i += blockDim.x) {
      const double v = st.Jab[i];
      if (v != 0.0) {
        atomicAdd(a.J + (size_t)(oa + i / NB) * nbf + ob + i % NB, v);
        st.Jab[i] = 0.0;
      }
    }
    for (int w = warp; w < nw; w += TPQ_STRIP_WARPS) {
      unsigned bits = st.touched[w];
      while (bits) {
        const int x = 32 * w + __ffs(bits) - 1;
        bits &= bits - 1;
        const int ox = __ldg(a.ao + x), nx = 2 * __ldg(a.shl + x) + 1;
        for (int e = lane; e < (NA + NB) * nx; e += 32) {
          const int row = e / nx, col = ox + e % nx;
          double* p = st.K + (size_t)row * nbf + col;
          const double v = *p;
          if (v != 0.0) {
            atomicAdd(a.K + (size_t)(row < NA ? oa + row : ob + row - NA) * nbf + col, v);
            *p = 0.0;
          }
        }
      }
      __syncwarp();
      if (lane == 0) st.touched[w] = 0u;
    }
    __syncthreads();
  }
}

}  // namespace mako
