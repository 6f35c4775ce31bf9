// eri_slab.cuh -- slot-batched DMMA kernel for the mid angular-momentum classes.
//
// PAPER.md Alg. 1 (L194-L213) with the striped->blocked layout change of S3.1.2 (L233-L249):
//   * a warp owns one bra pair and <= KT kets; the ket primitive pairs ("slots") of consecutive kets
//     are batched, NS at a time;
//   * R phase (striped, SL): lane c computes, fully in registers, the Boys seed and the Eq. 5
//     R-recursion of one primitive quartet (bra primitive ij, slot s) and stores R^{(0)} to a
//     warp-private SMEM row (the SL -> BL hand-off);
//   * GEMM1 (Eq. 7a) on FP64 DMMA with the slots flattened into N:
//       T1[ab][(s,q)] += sum_p E~_ab^{ij}[ab][p] R^{(ij,s)}_{p+q}
//     B fragments are gathered from the R rows through a per-CTA offset table, so [p|q]
//     (Eq. 6) is never materialised and there is no per-slot padding of nH_cd;
//   * GEMM2 (Eq. 7b / Eq. 11) per slot, chained in registers: the GEMM1 accumulator fragment is the
//     A operand; columns of other slots are masked through a zero B operand;
//   * the per-ket block (ab|cd) accumulates in warp SMEM and is digested (a9) when the ket completes.
#pragma once

#include "eri_core.cuh"
#include "eri_tpq.cuh"
#include "eri_kf.cuh"

namespace mako {

template <int X, int Y>
struct SlabCfg {
  using C = ClsXY<X, Y>;
  static constexpr int T1B = C::L >= 5 ? 32 : 40;  // accumulator budget (doubles / lane) for T1 + C2
  static constexpr int c2(int) { return C::MT * C::NT2 * 2; }
  static constexpr int t1(int ns) { return C::MT * ((ns * C::NHCD + 7) / 8) * 2; }
  static constexpr int pick_ns() {
    int ns = 16;
    while (ns > 1 && t1(ns) + c2(ns) > T1B) ns >>= 1;
    return ns;
  }
  static constexpr int NS = pick_ns();
  static constexpr int NT1B = (NS * C::NHCD + 7) / 8;
  static constexpr bool OK = C::L <= 6 && t1(NS) + c2(NS) <= 64;
  static constexpr int RSTRIDE = C::NH | 1;       // odd row stride (doubles)
  // CTA table: B-fragment offsets [KS1][NT1B][32] (slot << 10 | hermite index, 0xffff = zero; 16-bit: slot < 16)
  static constexpr int HOFS_INTS = C::KS1 * NT1B * 32;
  static_assert(NS <= 16 && C::NH < 1024, "16-bit B-fragment offsets");
  // warp SMEM (doubles): R rows (also the digestion partial-sum scratch), V for NS kets, J_ab partial, D
  // blocks, the ket-primitive list of the R super-batch (RCAP ints)
  static constexpr int w_r(int rcap) { return rcap * RSTRIDE; }
  static constexpr int W_V = NS * C::NAB * C::NCD;
  static constexpr int W_P = 2 * (C::NA + C::NB) * C::NCD;  // digestion partial sums (R rows outlive a batch)
  static constexpr int warp_dbl(int rcap) { return w_r(rcap) + W_V + C::NAB + 2 + C::W_D + (rcap + 1) / 2 + W_P; }
  static constexpr size_t smem(int rcap) {
    return ((sizeof(uint16_t) * HOFS_INTS + 15) / 16) * 16 + sizeof(double) * 4 * warp_dbl(rcap);
  }
  static constexpr bool fits4(int rcap) { return 4 * (smem(rcap) + 1024) <= 228 * 1024; }
  // R rows per warp = primitive quartets per R phase: one per lane (32) unless four CTAs (the register-bound
  // occupancy of these instantiations) would then not fit in shared memory
  static constexpr int RCAP = fits4(32) ? 32 : (fits4(24) ? 24 : 16);
  static constexpr int W_R = w_r(RCAP);
  static constexpr int WARP_DBL = warp_dbl(RCAP);
  static constexpr size_t SMEM = smem(RCAP);
};

template <int X, int Y>
constexpr bool use_slab() {
  // measured per class (profiles/README.md): only (pp|pp) and (dp|pp) -- bras with up to 16 primitive
  // pairs and pp kets -- still beat the warp-per-quartet kernel with its once-per-quartet R rows
  return !use_tpq(X, Y) && SlabCfg<X, Y>::OK && in_list(kSlabPick, X * 100 + Y);
}

// warp-per-quartet class run transposed: task pairs from the ket bucket Y, kets from X (jk_kernel<Y, X>
// evaluates (cd|ab) = (ab|cd) and digests it with the same six updates); its reduced tier runs
// jk_kernel_q<Y, X> likewise
template <int X, int Y>
constexpr bool use_jk_swap() {
  return X != Y && !use_tpq(X, Y) && !use_kf<X, Y>() && !use_kf_swap<X, Y>() && !use_slab<X, Y>() &&
         in_list(kJkSwapPick, X * 100 + Y);
}

template <int X, int Y, bool DW = false>
__global__ void __launch_bounds__(128, 4) slab_jk_kernel(JKArgs a) {
  using C = ClsXY<X, Y>;
  using S = SlabCfg<X, Y>;
  constexpr int NAB = C::NAB, NCD = C::NCD, NHAB = C::NHAB, NHCD = C::NHCD, L = C::L;
  constexpr int MT = C::MT, KS1 = C::KS1, NT2 = C::NT2, NS = S::NS, NT1B = S::NT1B, RS = S::RSTRIDE;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  uint16_t* hofs = reinterpret_cast<uint16_t*>(smem_raw);
  double* wbase = reinterpret_cast<double*>(smem_raw + ((sizeof(uint16_t) * S::HOFS_INTS + 15) / 16) * 16);
  // B-fragment offset table: lane (g,t), k-step ks, n-tile nt -> R row slot and Hermite index of p+q
  for (int o = threadIdx.x; o < S::HOFS_INTS; o += blockDim.x) {
    const int ln = o & 31, nt = (o >> 5) % NT1B, ks = (o >> 5) / NT1B;
    const int p = 4 * ks + (ln & 3), col = 8 * nt + (ln >> 2);
    int v = -1;
    if (p < NHAB && col < NS * NHCD) {
      const int s = col / NHCD, q = col % NHCD;
      int t1, u1, v1, t2, u2, v2;
      hdecode(p, t1, u1, v1);
      hdecode(q, t2, u2, v2);
      v = (s << 10) | hidx(t1 + t2, u1 + u2, v1 + v2);
    }
    hofs[o] = (uint16_t)(v & 0xffff);
  }
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int g = lane >> 2, t = lane & 3;
  double* Rs = wbase + (size_t)warp * S::WARP_DBL;
  double* Vs = Rs + S::W_R;
  double* jab = Vs + S::W_V;
  int* skl = reinterpret_cast<int*>(jab + NAB + 2 + C::W_D);  // ket primitive of each super-batch slot
  double* Ps = jab + NAB + 2 + C::W_D + (S::RCAP + 1) / 2;     // digestion scratch
  for (int i = lane; i < S::W_R; i += 32) Rs[i] = 0.0;  // unused slots must stay finite
  __syncthreads();
  for (;;) {
  long long tg0, tg1;
  if (!grab_tasks(a, lane, tg0, tg1)) break;
  int U = find_entry(a, tg0);
  for (long long task = tg0; task < tg1; ++task) {
    while (__ldg(a.task_off + U + 1) <= task) ++U;
    const int P = __ldg(a.ent_P + U);
    const int r0 = __ldg(a.kbeg + U) + (int)(task - __ldg(a.task_off + U)) * a.KT;
    const int r1 = min(r0 + a.KT, __ldg(a.kend + U));
    const double QP = __ldg(a.bra.Q + P);
    const int sa = __ldg(a.bra.shA + P), sb = __ldg(a.bra.shB + P);
    const int oa = __ldg(a.ao + sa), ob = __ldg(a.ao + sb);
    const int b0 = __ldg(a.bra.poff + P), b1 = __ldg(a.bra.poff + P + 1);
    const int KAB = b1 - b0;
    const int nsl = max(1, min(NS, S::RCAP / KAB));  // slots per batch so that KAB * nsl <= RCAP R rows
    // super-batched R phase (KAB <= RCAP): the R rows of the next RCAP / KAB slots (all their bra
    // primitives) are computed in one pass, one primitive quartet per lane, and consumed by several GEMM
    // batches of <= nsl slots; with few bra primitives a batch alone would keep only KAB * nsl lanes busy
    const bool sup = KAB <= S::RCAP;
    int sb_left = 0, slot_base = 0;
    for (int i = lane; i < NAB; i += 32) jab[i] = 0.0;
    // ket cursor: ket r, next primitive kl
    int r = r0, kl = (r < r1) ? __ldg(a.ket.poff + r) : 0;
    while (r < r1) {
      if (sup && sb_left == 0) {
        // slots of the super-batch: the next RCAP / KAB ket primitives of surviving kets from the cursor
        const int nsup = S::RCAP / KAB;
        int rr = r, kk = kl, n = 0;
        while (n < nsup && rr < r1) {
          const double QQ = QP * __ldg(a.ket.Q + rr);
          if (QQ < a.thresh || !dw_keep<DW>(a, QQ, sa, sb, __ldg(a.ket.shA + rr), __ldg(a.ket.shB + rr))) {
            ++rr;
            if (rr < r1) kk = __ldg(a.ket.poff + rr);
            continue;
          }
          const int kend = __ldg(a.ket.poff + rr + 1);
          while (n < nsup && kk < kend) {
            if (lane == 0) skl[n] = kk;
            ++n;
            ++kk;
          }
          if (kk == kend) {
            ++rr;
            if (rr < r1) kk = __ldg(a.ket.poff + rr);
          }
        }
        if (n == 0) break;
        __syncwarp();
        // R phase: combo c = slot * KAB + bra primitive, one primitive quartet per lane (striped layout)
        for (int c = lane; c < n * KAB; c += 32) {
          const int ij = b0 + c % KAB, klc = skl[c / KAB];
          double p, Px, Py, Pz;
          load_pdat(a.bra.pdat, ij, p, Px, Py, Pz);
          double q, Qx, Qy, Qz;
          load_pdat<true>(a.ket.pdat, klc, q, Qx, Qy, Qz);
          double Rr[nH(L)];
          r_regs<L>(p, Px, Py, Pz, q, Qx, Qy, Qz, a.boys, Rr);
          double* row = Rs + (size_t)c * RS;
#pragma unroll
          for (int h = 0; h < nH(L); ++h) row[h] = Rr[h];
        }
        __syncwarp();
        sb_left = n;
        slot_base = 0;
      }
      // ---- build a batch of up to nsl slots over consecutive kets (warp-uniform) ----
      int s_kl[NS], s_vk[NS];   // slot -> ket primitive, V row (ket within batch)
      int vk_r[NS];             // V row -> ket index
      bool vk_done[NS];
      int ns = 0, nvk = 0;
      const bool cont = kl != __ldg(a.ket.poff + r);  // batch starts inside a ket (V row carries over)
      const int nsl_b = sup ? min(nsl, sb_left) : nsl;
      while (ns < nsl_b && r < r1) {
        const double QQ = QP * __ldg(a.ket.Q + r);
        if (QQ < a.thresh || !dw_keep<DW>(a, QQ, sa, sb, __ldg(a.ket.shA + r), __ldg(a.ket.shB + r))) {
          ++r;
          if (r < r1) kl = __ldg(a.ket.poff + r);
          continue;
        }
        const int kend = __ldg(a.ket.poff + r + 1);
        vk_r[nvk] = r;
        while (ns < nsl_b && kl < kend) {
          s_kl[ns] = kl;
          s_vk[ns] = nvk;
          ++ns;
          ++kl;
        }
        vk_done[nvk] = (kl == kend);
        ++nvk;
        if (kl == kend) {
          ++r;
          if (r < r1) kl = __ldg(a.ket.poff + r);
        }
      }
      if (ns == 0) break;
      // zero V rows of kets starting in this batch (a continued ket keeps its partial block in row 0)
      for (int v = (cont ? 1 : 0); v < nvk; ++v)
        for (int i = lane; i < NAB * NCD; i += 32) Vs[v * NAB * NCD + i] = 0.0;
      // ---- R phase + GEMM1, bra primitives in chunks of ijn (ns * ijn <= RCAP R rows) ----
      double t1[MT][NT1B][2];
#pragma unroll
      for (int m = 0; m < MT; ++m)
#pragma unroll
        for (int n = 0; n < NT1B; ++n) t1[m][n][0] = t1[m][n][1] = 0.0;
      if (sup) {
        // GEMM1 over the super-batch rows of this batch's slots (slot_base ...)
        for (int ijl = 0; ijl < KAB; ++ijl) {
          const double* __restrict__ EA = a.bra.EbraD + (size_t)(b0 + ijl) * frag_a_doubles(C::LA, C::LB);
#pragma unroll
          for (int ks = 0; ks < KS1; ++ks) {
            double af[MT];
#pragma unroll
            for (int m = 0; m < MT; ++m) af[m] = __ldg(EA + (m * KS1 + ks) * 32 + lane);
#pragma unroll
            for (int n = 0; n < NT1B; ++n) {
              const int h = hofs[(ks * NT1B + n) * 32 + lane] == 0xffff ? -1 : hofs[(ks * NT1B + n) * 32 + lane];
              const double b =
                  (h >= 0 && (h >> 10) < ns) ? Rs[((slot_base + (h >> 10)) * KAB + ijl) * RS + (h & 1023)] : 0.0;
#pragma unroll
              for (int m = 0; m < MT; ++m) dmma884(t1[m][n][0], t1[m][n][1], af[m], b);
            }
          }
        }
        slot_base += ns;
        sb_left -= ns;
      } else {
      const int ijc = max(1, S::RCAP / ns);
        for (int ij0 = 0; ij0 < KAB; ij0 += ijc) {
          const int ijn = min(ijc, KAB - ij0);
          // R phase: combo c = s * ijn + (ij - ij0), one primitive quartet per lane (striped layout)
          const int ncombo = ns * ijn;
          for (int c = lane; c < ncombo; c += 32) {
            const int s = c / ijn, ij = b0 + ij0 + c % ijn;
            int klc = 0;
#pragma unroll
            for (int z = 0; z < NS; ++z)
              if (z == s) klc = s_kl[z];
            double p, Px, Py, Pz;
          load_pdat(a.bra.pdat, ij, p, Px, Py, Pz);
            double q, Qx, Qy, Qz;
          load_pdat<true>(a.ket.pdat, klc, q, Qx, Qy, Qz);
            double Rr[nH(L)];
            r_regs<L>(p, Px, Py, Pz, q, Qx, Qy, Qz, a.boys, Rr);
            double* row = Rs + (size_t)c * RS;
#pragma unroll
            for (int h = 0; h < nH(L); ++h) row[h] = Rr[h];
          }
          __syncwarp();
          // GEMM1 (blocked layout): T1[ab][(s,q)] += E~_ab^{ij} R^{(ij,s)}_{p+q}
          for (int ijl = 0; ijl < ijn; ++ijl) {
            const double* __restrict__ EA = a.bra.EbraD + (size_t)(b0 + ij0 + ijl) * frag_a_doubles(C::LA, C::LB);
#pragma unroll
            for (int ks = 0; ks < KS1; ++ks) {
              double af[MT];
#pragma unroll
              for (int m = 0; m < MT; ++m) af[m] = __ldg(EA + (m * KS1 + ks) * 32 + lane);
#pragma unroll
              for (int n = 0; n < NT1B; ++n) {
                const int h = hofs[(ks * NT1B + n) * 32 + lane] == 0xffff ? -1 : hofs[(ks * NT1B + n) * 32 + lane];
                const double b = (h >= 0 && (h >> 10) < ns) ? Rs[((h >> 10) * ijn + ijl) * RS + (h & 1023)] : 0.0;
#pragma unroll
                for (int m = 0; m < MT; ++m) dmma884(t1[m][n][0], t1[m][n][1], af[m], b);
              }
            }
          }
          __syncwarp();
        }
      }
      // ---- GEMM2 per slot (register chained), accumulate into the slot's ket row of V ----
      for (int s = 0; s < ns; ++s) {
        int kls = 0, vks = 0;
#pragma unroll
        for (int z = 0; z < NS; ++z)
          if (z == s) { kls = s_kl[z]; vks = s_vk[z]; }
        const double* __restrict__ Ek = a.ket.Eket + (size_t)kls * (NHCD * NCD);
        double c2[MT][NT2][2];
#pragma unroll
        for (int m = 0; m < MT; ++m)
#pragma unroll
          for (int n = 0; n < NT2; ++n) c2[m][n][0] = c2[m][n][1] = 0.0;
        const int c0 = s * NHCD, c1 = c0 + NHCD;
#pragma unroll
        for (int n = 0; n < NT1B; ++n) {
          if (8 * n >= c1 || 8 * n + 8 <= c0) continue;
#pragma unroll
          for (int e = 0; e < 2; ++e) {
            const int col = 8 * n + 2 * t + e;
            const bool in = col >= c0 && col < c1;
            const int qq = col - c0;
#pragma unroll
            for (int n2 = 0; n2 < NT2; ++n2) {
              const int cd = 8 * n2 + g;
              const double b = (in && cd < NCD) ? __ldg(Ek + qq * NCD + cd) : 0.0;
#pragma unroll
              for (int m = 0; m < MT; ++m) dmma884(c2[m][n2][0], c2[m][n2][1], t1[m][n][e], b);
            }
          }
        }
        double* Vr = Vs + (size_t)vks * (NAB * NCD);
#pragma unroll
        for (int m = 0; m < MT; ++m)
#pragma unroll
          for (int n2 = 0; n2 < NT2; ++n2)
#pragma unroll
            for (int i = 0; i < 2; ++i) {
              const int row = 8 * m + g, col = 8 * n2 + 2 * t + i;
              if (row < NAB && col < NCD) Vr[row * NCD + col] += c2[m][n2][i];
            }
        __syncwarp();
      }
      // ---- digest completed kets; an unfinished last ket is moved to row 0 for the next batch ----
      for (int v = 0; v < nvk; ++v) {
        if (!vk_done[v]) {
          if (v != 0)
            for (int i = lane; i < NAB * NCD; i += 32) Vs[i] = Vs[v * NAB * NCD + i];
          __syncwarp();
          continue;
        }
        const int R = vk_r[v];
        const int sc = __ldg(a.ket.shA + R), sd = __ldg(a.ket.shB + R);
        double deg = 1.0;
        if (sa == sb) deg *= 0.5;
        if (sc == sd) deg *= 0.5;
        if (a.same_bucket && P == R) deg *= 0.5;
        digest<C>(Vs + (size_t)v * NAB * NCD, deg, oa, ob, __ldg(a.ao + sc), __ldg(a.ao + sd), a.D, a.nbf, a.J, a.K,
                  jab, jab + NAB + 2, Ps, lane);
        __syncwarp();
      }
    }
    for (int ab = lane; ab < NAB; ab += 32)
      {  // J_ab block, oriented for contiguous runs (blk_rc, eri_core.cuh)
        int i, j;
        blk_rc<C::NA, C::NB>(ab, i, j);
        atomicAdd(a.J + blk_dst<C::NA, C::NB>(oa + i, ob + j, a.nbf), jab[i * C::NB + j]);
      }
    __syncwarp();
  }
  }
}

}  // namespace mako
