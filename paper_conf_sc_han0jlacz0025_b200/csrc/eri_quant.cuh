// eri_quant.cuh -- stage-aware reduced-precision tier of the warp-per-quartet kernel (SURVEY.md §8.f1,
// QuantMako, §3.2).
//
// Stages and their precision ("preserves high-precision arithmetic for the recursive
// integral generation step while introducing [reduced-precision] arithmetic into the basis
// transformation step"; L296 dual-stage accumulation):
//   a4 Boys, a5 R recursion         FP64 (compute_R), level 0 rounded once to TF32 (10-bit mantissa)
//   a7 GEMM1 [ab|q] = E~_AB [p|q]   mma.sync.m16n8k8 TF32 x TF32 -> FP32 accumulators (SASS HMMA.1688)
//   a8 GEMM2 (ab|cd) = [ab|q] E~_CD^T  GEMM1's FP32 accumulator fragment rounded to TF32 is GEMM2's A
//                                   fragment (chained in registers), FP32 accumulation over ket primitives
//   a9 digestion                    FP64 (the same `digest` as the FP64 tier)
// Operand format: TF32 instead of the paper's FP16 + per-class power-of-two scales (reading R19 in
// DESIGN.md): the same 10-bit mantissa (unit roundoff 2^-11), with FP32's 8-bit exponent, so the
// 10^20+ dynamic range of an R row (the (-2 rho)^n factors) needs no scaling and cannot overflow.
// Operands are stored in fragment order by pairs.cu (build_lowp_kernel): one 128-bit load per A
// fragment of GEMM1, one 64-bit load per B fragment of GEMM2, zero padding in storage.
//
// Per-stage error budget (unit roundoff u = 2^-11 per TF32 operand, v = 2^-24 per FP32 add):
//   GEMM1 term E~ R: <= 2u relative; FP32 sum over K1 = K_AB nH_ab terms: <= K1 v of sum|terms|
//   GEMM2 operands [ab|q] and E~_cd: <= 2u relative; FP32 sum over K2 = K_CD nH_cd terms: K2 v
//   => |d(ab|cd)| <= (4u + (K1 + K2) v) * S, S = sum_{p,q} |E~_ab[p]| |R_{p+q}| |E~_cd[q]|
//   (S >= |(ab|cd)|; it is what cancellation in the MMD sum leaves behind). Measured against the
//   oracle per class in tests/test_gpu_quant.py.
#pragma once

#include "eri_core.cuh"

namespace mako {

__device__ __forceinline__ unsigned f2tf32(float x) {
  unsigned r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
  return r;
}

__device__ __forceinline__ void mma_tf32(float (&c)[4], const float4& a, unsigned b0, unsigned b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};\n"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(__float_as_uint(a.x)), "r"(__float_as_uint(a.y)), "r"(__float_as_uint(a.z)), "r"(__float_as_uint(a.w)),
        "r"(b0), "r"(b1));
}
__device__ __forceinline__ void mma_tf32(float (&c)[4], unsigned a0, unsigned a1, unsigned a2, unsigned a3, unsigned b0,
                                         unsigned b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};\n"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

// class geometry of the TF32 tier (m16n8k8 tiles)
template <class C>
struct ClsQ {
  static constexpr int MT = (C::NAB + 15) / 16;   // m16 tiles over ab
  static constexpr int KS1 = (C::NHAB + 7) / 8;   // GEMM1 k8 steps over p
  static constexpr int NT1 = (C::NHCD + 7) / 8;   // GEMM1 n8 tiles over q (= GEMM2 k8 steps)
  static constexpr int NT2 = (C::NCD + 7) / 8;    // GEMM2 n8 tiles over cd
#ifndef MAKO_QREGB_HI
#define MAKO_QREGB_HI 96
#endif
#ifndef MAKO_QREGB_LO
#define MAKO_QREGB_LO 72
#endif
  static constexpr int REGB = C::L >= 8 ? MAKO_QREGB_HI : MAKO_QREGB_LO;  // FP32 accumulators per lane
  static constexpr int MCMAX = clampi(REGB / (4 * (NT1 + NT2)), 1, MT);
  static constexpr int NCHUNK = (MT + MCMAX - 1) / MCMAX;
  static constexpr int MC = (MT + NCHUNK - 1) / NCHUNK;
  static constexpr int A_FL = MT * KS1 * 128;     // = lowp_a_floats of the bra bucket
  static constexpr int B_FL = NT1 * NT2 * 64;     // = lowp_b_floats of the ket bucket
  static constexpr int W_R32 = (C::KR * C::NH + 1) / 2;  // TF32 R rows (in doubles)
  static constexpr int WARP_DBL = C::WARP_DBL + W_R32;
};

// (ab|cd) block, TF32 tier: same dataflow as quartet_block (eri_core.cuh), m16n8k8 fragments
// (lane = 4g + t): A[g|g+8][t|t+4]; B[k=t|t+4][n=g]; C[g|g+8][2t|2t+1].  GEMM2 takes its k index in
// the permuted order slot t <-> q = 8nt+2t, slot t+4 <-> q = 8nt+2t+1, so that GEMM1's accumulator
// fragment is GEMM2's A fragment without any data movement.
template <class C>
__device__ void quartet_block_q(const PairView& bra, int P, const PairView& ket, int R, double* __restrict__ Rbuf,
                                float* __restrict__ R32, double* __restrict__ V, const uint16_t* __restrict__ htab,
                                const uint32_t* __restrict__ rtab, const double* __restrict__ btab, int lane) {
  using Q = ClsQ<C>;
  constexpr int KR = C::KR, NH = C::NH;
  constexpr bool ONECHUNK = Q::NCHUNK == 1;
  constexpr bool STREAM = Q::NCHUNK == 1 && KR == 1;
  const int g = lane >> 2, t = lane & 3;
  const int b0 = __ldg(bra.poff + P), b1 = __ldg(bra.poff + P + 1);
  const int k0 = __ldg(ket.poff + R), k1 = __ldg(ket.poff + R + 1);
  if constexpr (!ONECHUNK)
    for (int i = lane; i < C::NAB * C::NCD; i += 32) V[i] = 0.0;
  float c2[Q::MC][Q::NT2][4];
#pragma unroll
  for (int mc = 0; mc < Q::MC; ++mc)
#pragma unroll
    for (int n2 = 0; n2 < Q::NT2; ++n2) c2[mc][n2][0] = c2[mc][n2][1] = c2[mc][n2][2] = c2[mc][n2][3] = 0.f;
  for (int kl = k0; kl < k1; ++kl) {
    double q, Qx, Qy, Qz;
    load_pdat(ket.pdat, kl, q, Qx, Qy, Qz);
    const float2* __restrict__ Ek = reinterpret_cast<const float2*>(ket.EketF + (size_t)kl * Q::B_FL) + lane;
    float t1s[Q::MC][Q::NT1][4];
    if constexpr (STREAM) {
#pragma unroll
      for (int mc = 0; mc < Q::MC; ++mc)
#pragma unroll
        for (int nt = 0; nt < Q::NT1; ++nt) t1s[mc][nt][0] = t1s[mc][nt][1] = t1s[mc][nt][2] = t1s[mc][nt][3] = 0.f;
    }
    for (int ig0 = b0; ig0 < b1; ig0 += KR) {
      const int ign = min(KR, b1 - ig0);
      for (int il = 0; il < ign; ++il) {
        double p, Px, Py, Pz;
        load_pdat(bra.pdat, ig0 + il, p, Px, Py, Pz);
        compute_R<C, true>(p, Px, Py, Pz, q, Qx, Qy, Qz, Rbuf, Rbuf + NH, rtab, btab, lane, R32 + il * NH);
      }
      for (int ch = 0; ch < Q::NCHUNK; ++ch) {
        float t1[Q::MC][Q::NT1][4];
#pragma unroll
        for (int mc = 0; mc < Q::MC; ++mc)
#pragma unroll
          for (int nt = 0; nt < Q::NT1; ++nt)
#pragma unroll
            for (int i = 0; i < 4; ++i) t1[mc][nt][i] = STREAM ? t1s[mc][nt][i] : 0.f;
        for (int il = 0; il < ign; ++il) {
          const float4* __restrict__ E =
              reinterpret_cast<const float4*>(bra.EbraF + (size_t)(ig0 + il) * Q::A_FL) + lane;
          const float* __restrict__ Rr = R32 + il * NH;
#pragma unroll
          for (int ks = 0; ks < Q::KS1; ++ks) {
            const int p0 = 8 * ks + t, p1 = p0 + 4;
            float4 a[Q::MC];
#pragma unroll
            for (int mc = 0; mc < Q::MC; ++mc) {
              const int mt = ch * Q::MC + mc;
              a[mc] = mt < Q::MT ? __ldg(E + (mt * Q::KS1 + ks) * 32) : make_float4(0.f, 0.f, 0.f, 0.f);
            }
#pragma unroll
            for (int nt = 0; nt < Q::NT1; ++nt) {
              const int qc = 8 * nt + g;
              const bool qok = qc < C::NHCD;
              const unsigned bb0 = (qok && p0 < C::NHAB) ? __float_as_uint(Rr[htab[p0 * C::NHCD + qc]]) : 0u;
              const unsigned bb1 = (qok && p1 < C::NHAB) ? __float_as_uint(Rr[htab[p1 * C::NHCD + qc]]) : 0u;
#pragma unroll
              for (int mc = 0; mc < Q::MC; ++mc)
                if (ch * Q::MC + mc < Q::MT) mma_tf32(t1[mc][nt], a[mc], bb0, bb1);
            }
          }
        }
        if constexpr (STREAM) {
#pragma unroll
          for (int mc = 0; mc < Q::MC; ++mc)
#pragma unroll
            for (int nt = 0; nt < Q::NT1; ++nt)
#pragma unroll
              for (int i = 0; i < 4; ++i) t1s[mc][nt][i] = t1[mc][nt][i];
          if (ig0 + KR < b1) continue;
        }
        if constexpr (!ONECHUNK) {
#pragma unroll
          for (int mc = 0; mc < Q::MC; ++mc)
#pragma unroll
            for (int n2 = 0; n2 < Q::NT2; ++n2) c2[mc][n2][0] = c2[mc][n2][1] = c2[mc][n2][2] = c2[mc][n2][3] = 0.f;
        }
        // GEMM2: A fragment (rows g|g+8, slots t|t+4) = (c0, c2, c1, c3) of GEMM1's n-tile nt
#pragma unroll
        for (int nt = 0; nt < Q::NT1; ++nt) {
          unsigned af[Q::MC][4];
#pragma unroll
          for (int mc = 0; mc < Q::MC; ++mc) {
            af[mc][0] = f2tf32(t1[mc][nt][0]);
            af[mc][1] = f2tf32(t1[mc][nt][2]);
            af[mc][2] = f2tf32(t1[mc][nt][1]);
            af[mc][3] = f2tf32(t1[mc][nt][3]);
          }
#pragma unroll
          for (int n2 = 0; n2 < Q::NT2; ++n2) {
            const float2 b = __ldg(Ek + (nt * Q::NT2 + n2) * 32);
#pragma unroll
            for (int mc = 0; mc < Q::MC; ++mc)
              if (ch * Q::MC + mc < Q::MT)
                mma_tf32(c2[mc][n2], af[mc][0], af[mc][1], af[mc][2], af[mc][3], __float_as_uint(b.x),
                         __float_as_uint(b.y));
          }
        }
        if constexpr (!ONECHUNK) {
#pragma unroll
          for (int mc = 0; mc < Q::MC; ++mc)
#pragma unroll
            for (int n2 = 0; n2 < Q::NT2; ++n2)
#pragma unroll
              for (int i = 0; i < 4; ++i) {
                const int row = 16 * (ch * Q::MC + mc) + g + 8 * (i >> 1), col = 8 * n2 + 2 * t + (i & 1);
                if (row < C::NAB && col < C::NCD) V[row * C::NCD + col] += (double)c2[mc][n2][i];
              }
        }
      }
      __syncwarp();  // R rows are overwritten by the next bra-primitive group
    }
  }
  if constexpr (ONECHUNK) {
#pragma unroll
    for (int mc = 0; mc < Q::MC; ++mc)
#pragma unroll
      for (int n2 = 0; n2 < Q::NT2; ++n2)
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int row = 16 * mc + g + 8 * (i >> 1), col = 8 * n2 + 2 * t + (i & 1);
          if (row < C::NAB && col < C::NCD) V[row * C::NCD + col] = (double)c2[mc][n2][i];
        }
  }
  __syncwarp();
}

}  // namespace mako
