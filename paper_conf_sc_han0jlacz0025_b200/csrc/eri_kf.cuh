// eri_kf.cuh -- "ket-first" kernel for classes with a light ket (ss, ps, pp, ds) and a heavier bra.
//
// Eq. 7 evaluated in the cheaper order for n_cd << n_ab, with the two stages on
// the two separate FP64 pipes of sm_100a (S6: DFMA and DMMA run concurrently):
//   DFMA (per lane, registers):  W^{ij}[p][cd] = sum_kl sum_q R^{(ij,kl)}_{p+q} (-1)^{|q|} E~_cd^{kl}[q][cd]
//                                (Boys a4 + Eq. 5 a5 + the ket contraction, a striped layout: lanes own kets)
//   DMMA (warp, mma.sync f64):   V[ab][(k,cd)] += sum_p E~_ab^{ij}[ab][p] W^{ij}[p][(k,cd)]
//                                (the bra contraction as one GEMM with N = kets x cd; the blocked layout of
//                                L233-L249 is the SMEM hand-off of W)
// A warp owns one bra pair and NK kets; 32/NK lanes share a ket and split its p range (each lane
// recomputes the ket's R -- cheaper than synchronising).  Digestion (a9) is spread over the lanes of
// each ket; J_ab is reduced across kets with warp shuffles.
#pragma once

#include "eri_core.cuh"
#include "eri_tpq.cuh"

namespace mako {

template <int X, int Y>
struct KfCfg {
  using C = ClsXY<X, Y>;
  static constexpr int vfr(int nk) { return C::MT * ((nk * C::NCD + 7) / 8) * 2; }
  static constexpr int wpart(int nk) { return ((C::NHAB + (32 / nk) - 1) / (32 / nk)) * C::NCD; }
  static constexpr int regs(int nk) { return nH(C::L) + wpart(nk) + vfr(nk); }
  static constexpr int pick() {
    return (vfr(16) <= 24 && regs(16) <= 128)  ? 16
           : (vfr(8) <= 24 && regs(8) <= 128)  ? 8
           : (vfr(4) <= 24 && regs(4) <= 128)  ? 4
           : (vfr(2) <= 24 && regs(2) <= 136)  ? 2
                                               : 0;
  }
  static constexpr int NK = pick();                      // kets per warp task
  static constexpr int LPK = NK ? 32 / NK : 1;           // lanes per ket
  static constexpr int PP = (C::NHAB + LPK - 1) / LPK;   // p values per lane
  static constexpr int NTV = (NK * C::NCD + 7) / 8;      // n8 tiles of V / W columns
  static constexpr int COLS = NTV * 8;
  static constexpr int WS = COLS + ((4 - COLS % 16) + 16) % 16;  // row stride = 4 (mod 16): conflict-free B loads
  static constexpr int ROWS = (C::MT * 8 > C::KS1 * 4) ? C::MT * 8 : C::KS1 * 4;
  static constexpr int WARP_DBL = ROWS * WS;
  // per-ket D slots (D_cd | D_bd | D_bc | D_ad | D_ac, odd stride) + per-warp D_ab, filled by cp.async
  static constexpr int OCD = 0, OBD = OCD + C::NCD, OBC = OBD + C::NB * C::ND, OAD = OBC + C::NB * C::NC,
                       OAC = OAD + C::NA * C::ND, NDK = OAC + C::NA * C::NC, NDKS = NDK | 1;
  static constexpr int WARP_D = (NK > 0 ? NK : 1) * NDKS + C::NAB;
  static constexpr size_t SMEM = sizeof(double) * 4 * (WARP_DBL + WARP_D);
  static constexpr bool OK = NK > 0 && C::NHCD * C::NCD <= 140 && C::L <= 6;
  // 3 CTAs/SM (<= 168 registers, some spills) measured faster for these instantiations, else no cap
  static constexpr int MINB = in_list(kKfCap3, X * 100 + Y) ? 3 : 1;
};

template <int X, int Y>
constexpr bool use_kf() {
  // measured per class on the valinomycin-sized workload (profiles/README.md): KF wins for light kets
  // with a heavier bra; pp kets (8-fold redundant R per ket) stay on the slot-batched kernel
  return KfCfg<X, Y>::OK && in_list(kKfPick, X * 100 + Y);
}

// Transposed execution of class (X|Y), X > Y: the task pair comes from bucket Y and the lanes take
// pairs of bucket X, i.e. kf_jk_kernel<Y, X> computes (cd|ab) = (ab|cd) (8-fold symmetry) with the
// lighter side contracted per lane.  Used when the canonical ket has more functions than the bra.
template <int X, int Y>
constexpr bool use_kf_swap() {
  if constexpr (X != Y) return KfCfg<Y, X>::OK && in_list(kKfSwapPick, X * 100 + Y);
  return false;
}

template <int X, int Y, bool DW>
__device__ __forceinline__ void kf_body(const JKArgs& a);
template <int X, int Y, bool DW = false>
__global__ void __launch_bounds__(128) kf_kernel_free(JKArgs a) { kf_body<X, Y, DW>(a); }
template <int X, int Y, bool DW = false>
__global__ void __launch_bounds__(128, 3) kf_kernel_capped(JKArgs a) { kf_body<X, Y, DW>(a); }
template <int X, int Y, bool DW = false>
constexpr auto kf_jk_kernel_ptr() {
  if constexpr (KfCfg<X, Y>::MINB > 1) return &kf_kernel_capped<X, Y, DW>;
  else return &kf_kernel_free<X, Y, DW>;
}

template <int X, int Y, bool DW>
__device__ __forceinline__ void kf_body(const JKArgs& a) {
  using C = ClsXY<X, Y>;
  using K = KfCfg<X, Y>;
  constexpr int NAB = C::NAB, NCD = C::NCD, NHAB = C::NHAB, NHCD = C::NHCD, L = C::L;
  constexpr int NA = C::NA, NB = C::NB, NC = C::NC, ND = C::ND;
  constexpr int MT = C::MT, KS1 = C::KS1, NK = K::NK, LPK = K::LPK, PP = K::PP, NTV = K::NTV, WS = K::WS;
  extern __shared__ __align__(16) double kf_smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int g = lane >> 2, t = lane & 3;
  const int kk = lane / LPK, hh = lane % LPK;
  double* Ws = kf_smem + (size_t)warp * K::WARP_DBL;
  double* Dk = kf_smem + (size_t)4 * K::WARP_DBL + (size_t)warp * K::WARP_D + kk * K::NDKS;  // my ket's D slots
  double* Dab_s = kf_smem + (size_t)4 * K::WARP_DBL + (size_t)warp * K::WARP_D + NK * K::NDKS;
  for (int i = lane; i < K::WARP_DBL; i += 32) Ws[i] = 0.0;  // padding rows/cols stay zero forever
  __syncwarp();
  for (;;) {
  long long tg0, tg1;
  if (!grab_tasks(a, lane, tg0, tg1)) break;
  int U = find_entry(a, tg0);
  for (long long task = tg0; task < tg1; ++task) {
    while (__ldg(a.task_off + U + 1) <= task) ++U;
    const int P = __ldg(a.ent_P + U);
    const int r0 = __ldg(a.kbeg + U) + (int)(task - __ldg(a.task_off + U)) * NK;
    const int r1 = min(r0 + NK, __ldg(a.kend + U));
    const int R = r0 + kk;
    const double QP = __ldg(a.bra.Q + P);
    const double QQ = QP * __ldg(a.ket.Q + min(R, r1 - 1));
    const int sa = __ldg(a.bra.shA + P), sb = __ldg(a.bra.shB + P);
    const bool active = R < r1 && QQ >= a.thresh &&
                        dw_keep<DW>(a, QQ, sa, sb, __ldg(a.ket.shA + min(R, r1 - 1)), __ldg(a.ket.shB + min(R, r1 - 1)));
    const int oa = __ldg(a.ao + sa), ob = __ldg(a.ao + sb);
    const int b0 = __ldg(a.bra.poff + P), b1 = __ldg(a.bra.poff + P + 1);
    const int k0 = active ? __ldg(a.ket.poff + R) : 0, k1 = active ? __ldg(a.ket.poff + R + 1) : 0;
    const int sc = active ? __ldg(a.ket.shA + R) : 0, sd = active ? __ldg(a.ket.shB + R) : 0;
    const int oc = active ? __ldg(a.ao + sc) : 0, od = active ? __ldg(a.ao + sd) : 0;
    {
      // D sub-blocks of this task's quartets: asynchronous copies, waited for before the digestion
      const size_t nb = (size_t)a.nbf;
      for (int x = lane; x < NAB; x += 32) cp_async8(Dab_s + x, a.D + (oa + x / NB) * nb + ob + x % NB);
      if (active)
        for (int x = hh; x < K::NDK; x += LPK) {
          int r, c;
          if (x < K::OBD) { r = oc + x / ND; c = od + x % ND; }
          else if (x < K::OBC) { r = ob + (x - K::OBD) / ND; c = od + (x - K::OBD) % ND; }
          else if (x < K::OAD) { r = ob + (x - K::OBC) / NC; c = oc + (x - K::OBC) % NC; }
          else if (x < K::OAC) { r = oa + (x - K::OAD) / ND; c = od + (x - K::OAD) % ND; }
          else { r = oa + (x - K::OAC) / NC; c = oc + (x - K::OAC) % NC; }
          cp_async8(Dk + x, a.D + (size_t)r * nb + c);
        }
      cp_async_commit();
    }
    double vf[MT][NTV][2];
#pragma unroll
    for (int m = 0; m < MT; ++m)
#pragma unroll
      for (int n = 0; n < NTV; ++n) vf[m][n][0] = vf[m][n][1] = 0.0;
    for (int ij = b0; ij < b1; ++ij) {
      // ---- DFMA stage: this lane's p-slice of W^{ij} for its ket ----
      double p, Px, Py, Pz;
        load_pdat(a.bra.pdat, ij, p, Px, Py, Pz);
      double W[PP][NCD];
#pragma unroll
      for (int i = 0; i < PP; ++i)
#pragma unroll
        for (int j = 0; j < NCD; ++j) W[i][j] = 0.0;
      for (int kl = k0; kl < k1; ++kl) {
        double q, Qx, Qy, Qz;
        load_pdat<true>(a.ket.pdat, kl, q, Qx, Qy, Qz);
        double Rr[nH(L)];
        r_regs<L>(p, Px, Py, Pz, q, Qx, Qy, Qz, a.boys, Rr);
        const double* __restrict__ ek = a.ket.Eket + (size_t)kl * (NHCD * NCD);
        static_for<0, LPK>([&](auto hc) {
          constexpr int H = decltype(hc)::value;
          constexpr int p0 = H * PP, p1 = (p0 + PP < NHAB) ? p0 + PP : NHAB;
          if (hh == H) {
            static_for<0, NHCD>([&](auto qc) {
              constexpr int qq = decltype(qc)::value;
              double e[NCD];
#pragma unroll
              for (int j = 0; j < NCD; ++j) e[j] = __ldg(ek + qq * NCD + j);
              static_for<p0, p1>([&](auto pc) {
                constexpr int pp = decltype(pc)::value;
                constexpr int hs = h_sum(pp, qq);
#pragma unroll
                for (int j = 0; j < NCD; ++j) W[pp - p0][j] = fma(Rr[hs], e[j], W[pp - p0][j]);
              });
            });
          }
        });
      }
      // SL -> BL hand-off: W slice to SMEM row p, column (ket, cd)
#pragma unroll
      for (int i = 0; i < PP; ++i) {
        const int pr = hh * PP + i;
        if (pr < NHAB)
#pragma unroll
          for (int j = 0; j < NCD; ++j) Ws[pr * WS + kk * NCD + j] = W[i][j];
      }
      __syncwarp();
      // ---- DMMA stage: V[ab][(k,cd)] += E~_ab^{ij} W ----
      const double* __restrict__ EA = a.bra.EbraD + (size_t)ij * frag_a_doubles(C::LA, C::LB);  // A fragments
#pragma unroll
      for (int ks = 0; ks < KS1; ++ks) {
        const int pc = 4 * ks + t;
        double af[MT];
#pragma unroll
        for (int m = 0; m < MT; ++m) af[m] = __ldg(EA + (m * KS1 + ks) * 32 + lane);
#pragma unroll
        for (int n = 0; n < NTV; ++n) {
          const double b = Ws[pc * WS + 8 * n + g];
#pragma unroll
          for (int m = 0; m < MT; ++m) dmma884(vf[m][n][0], vf[m][n][1], af[m], b);
        }
      }
      __syncwarp();
    }
    // ---- V fragments to SMEM (rows ab, columns (k, cd)) ----
#pragma unroll
    for (int m = 0; m < MT; ++m)
#pragma unroll
      for (int n = 0; n < NTV; ++n)
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int row = 8 * m + g, col = 8 * n + 2 * t + i;
          if (row < NAB && col < NK * NCD) Ws[row * WS + col] = vf[m][n][i];
        }
    __syncwarp();
    // ---- digestion (a9) ----
    double deg = 1.0;
    if (sa == sb) deg *= 0.5;
    if (sc == sd) deg *= 0.5;
    if (a.same_bucket && P == R) deg *= 0.5;
    if (!active) deg = 0.0;
    const size_t nb = (size_t)a.nbf;
    const double* Vk = Ws + kk * NCD;  // V[ab][cd] of my ket = Vk[ab * WS + cd]
    cp_async_wait_all();
    __syncwarp();
    // J_ab: lanes with the same hh share ab; reduce over the kets
    for (int i0 = 0; i0 < NAB; i0 += LPK) {
      const int ab = i0 + hh;
      double s = 0.0;
      if (active && ab < NAB) {
#pragma unroll
        for (int x = 0; x < NCD; ++x) s = fma(Vk[ab * WS + x], Dk[K::OCD + x], s);
      }
      s *= deg;
#pragma unroll
      for (int o = LPK; o < 32; o <<= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
      if (kk == 0 && ab < NAB) atomicAdd(a.J + (oa + ab / NB) * nb + ob + ab % NB, 2.0 * s);
    }
    if (active) {
      // J_cd
      for (int cd = hh; cd < NCD; cd += LPK) {
        double s = 0.0;
#pragma unroll
        for (int ij = 0; ij < NAB; ++ij) s = fma(Vk[ij * WS + cd], Dab_s[ij], s);
        atomicAdd(a.J + (oc + cd / ND) * nb + od + cd % ND, 2.0 * deg * s);
      }
      // K_ac (NA*NC) | K_ad (NA*ND) | K_bc (NB*NC) | K_bd (NB*ND), flattened over the lanes of the ket
      constexpr int N1 = NA * NC, N2 = N1 + NA * ND, N3 = N2 + NB * NC, N4 = N3 + NB * ND;
      for (int x = hh; x < N4; x += LPK) {
        double s = 0.0;
        // (each block in the orientation with contiguous runs over consecutive lanes: blk_rc, eri_core.cuh)
        if (x < N1) {
          int i, k;
          blk_rc<NA, NC>(x, i, k);
          for (int j = 0; j < NB; ++j)
            for (int l = 0; l < ND; ++l) s = fma(Vk[(i * NB + j) * WS + k * ND + l], Dk[K::OBD + j * ND + l], s);
          atomicAdd(a.K + blk_dst<NA, NC>(oa + i, oc + k, a.nbf), deg * s);
        } else if (x < N2) {
          int i, l;
          blk_rc<NA, ND>(x - N1, i, l);
          for (int j = 0; j < NB; ++j)
            for (int k = 0; k < NC; ++k) s = fma(Vk[(i * NB + j) * WS + k * ND + l], Dk[K::OBC + j * NC + k], s);
          atomicAdd(a.K + blk_dst<NA, ND>(oa + i, od + l, a.nbf), deg * s);
        } else if (x < N3) {
          int j, k;
          blk_rc<NB, NC>(x - N2, j, k);
          for (int i = 0; i < NA; ++i)
            for (int l = 0; l < ND; ++l) s = fma(Vk[(i * NB + j) * WS + k * ND + l], Dk[K::OAD + i * ND + l], s);
          atomicAdd(a.K + blk_dst<NB, NC>(ob + j, oc + k, a.nbf), deg * s);
        } else {
          int j, l;
          blk_rc<NB, ND>(x - N3, j, l);
          for (int i = 0; i < NA; ++i)
            for (int k = 0; k < NC; ++k) s = fma(Vk[(i * NB + j) * WS + k * ND + l], Dk[K::OAC + i * NC + k], s);
          atomicAdd(a.K + blk_dst<NB, ND>(ob + j, od + l, a.nbf), deg * s);
        }
      }
    }
    __syncwarp();
  }
  }
}

}  // namespace mako
