// eri_kernels.cuh -- per-class kernels (J/K build, batch store, Schwarz diagonal) and launchers.
// Included with MAKO_DEFINE_KERNELS by the eri_cls_*.cu translation units (one per bra bucket),
// without it by the dispatcher (declarations only).
#pragma once

#include "mako_state.h"

namespace mako {

constexpr int CTA_THREADS = 128;
constexpr int CTA_WARPS = CTA_THREADS / 32;

template <int X, int Y>
mako_status launch_jk_xy(const JKArgs& a, void* stream, int* nlaunch);
template <int X, int Y>
mako_status launch_batch_xy(const BatchArgs& a, void* stream);
template <int X, int Y>
int jk_blocks_per_sm();
template <int X, int Y>
int task_kets_xy();
template <int X, int Y>
bool swap_xy();
template <int X, int Y>
bool lowp_xy();

}  // namespace mako

#ifdef MAKO_DEFINE_KERNELS
#include <algorithm>
#include <cstdlib>

#include "eri_core.cuh"
#include "eri_tpq.cuh"
#include "eri_slab.cuh"
#include "eri_kf.cuh"
#include "eri_quant.cuh"

namespace mako {

// classes with a reduced-precision (TF32) tier kernel: the warp-per-quartet DMMA family, where the
// basis transformation (GEMM1/GEMM2) dominates (the lane-per-ket, ket-first and
// slab families run the FP64 kernel in both tiers)
// Restricted to l <= 3 classes with n_ab >= 9 and L >= 6: measured per class (S6), the
// TF32 tier gains nothing where a 16-row tile is half empty (fs bras) or the R recursion dominates
// (L < 6), and the l = 4 classes ran slower in it.
template <int X, int Y>
constexpr bool has_lowp() {
  using C = ClsXY<X, Y>;
  return !use_tpq(X, Y) && !use_kf<X, Y>() && !use_kf_swap<X, Y>() && !use_slab<X, Y>() && C::LA <= 3 &&
         C::LC <= 3 && C::NAB >= 9 && C::L >= 6;
}

template <int X, int Y>
using JkCls = ClsXY<(use_jk_swap<X, Y>() ? Y : X), (use_jk_swap<X, Y>() ? X : Y)>;

// warps per CTA of the warp-per-quartet kernels: 4, fewer when the per-warp SMEM of a class does
// not fit (l = 4 classes: (gg|gg) runs 2 warps per CTA)
constexpr size_t SMEM_CTA_MAX = 227 * 1024 - 1024;
template <class C, int WD>
__host__ __device__ constexpr int warps_for() {
  constexpr size_t w = (SMEM_CTA_MAX - C::HTAB_BYTES - C::RTAB_BYTES) / (sizeof(double) * WD);
  static_assert(w >= 1, "class does not fit in shared memory");
  return w >= CTA_WARPS ? CTA_WARPS : (int)w;
}
template <class C>
__host__ __device__ constexpr int jk_warps() { return warps_for<C, C::WARP_DBL>(); }
template <class C>
__host__ __device__ constexpr size_t cta_smem_bytes() {
  return (size_t)C::HTAB_BYTES + C::RTAB_BYTES + sizeof(double) * (size_t)jk_warps<C>() * C::WARP_DBL;
}

// occupancy cap (4 CTAs/SM, <= 128 registers) measured faster for the fd-bra classes, (fp|dd), and (round 2,
// codes of the evaluated orientation) the transposed (fd|dp) (ff|pp) (ff|fs); (fd|fd) runs uncapped
template <int X, int Y>
constexpr int jk_minb() {
  return in_list(kJkCap4, X * 100 + Y) ? 4 : 1;
}

// Persistent J/K kernel: each warp pulls tasks (bra pair, <= KT consecutive kets) from a global counter.
// (An explicit minBlocks of 1 changes ptxas' register heuristic, so the cap is a separate wrapper.)
template <int X, int Y, bool DW>
__device__ __forceinline__ void jk_body(const JKArgs& a);
template <int X, int Y, bool DW = false>
__global__ void __launch_bounds__(CTA_THREADS) jk_kernel_free(JKArgs a) { jk_body<X, Y, DW>(a); }
template <int X, int Y, bool DW = false>
__global__ void __launch_bounds__(CTA_THREADS, 4) jk_kernel_capped(JKArgs a) { jk_body<X, Y, DW>(a); }
template <int X, int Y, bool DW = false>
constexpr auto jk_kernel_ptr() {
  if constexpr (jk_minb<X, Y>() > 1) return &jk_kernel_capped<X, Y, DW>;
  else return &jk_kernel_free<X, Y, DW>;
}

template <int X, int Y, bool DW>
__device__ __forceinline__ void jk_body(const JKArgs& a) {
  using C = ClsXY<X, Y>;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  uint16_t* htab = reinterpret_cast<uint16_t*>(smem_raw);
  uint32_t* rtab = reinterpret_cast<uint32_t*>(smem_raw + C::HTAB_BYTES);
  double* wbase = reinterpret_cast<double*>(smem_raw + C::HTAB_BYTES + C::RTAB_BYTES);
  init_tables<C>(htab, rtab);
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  double* Rbuf = wbase + (size_t)warp * C::WARP_DBL;
  double* V = Rbuf + C::W_R;
  double* jab = V + C::W_V;
  for (;;) {
  long long tg0, tg1;
  if (!grab_tasks(a, lane, tg0, tg1)) break;
  int U = find_entry(a, tg0);
  for (long long task = tg0; task < tg1; ++task) {
    while (__ldg(a.task_off + U + 1) <= task) ++U;
    const int P = __ldg(a.ent_P + U);
    const int r0 = __ldg(a.kbeg + U) + (int)(task - __ldg(a.task_off + U)) * a.KT;
    const int r1 = min(r0 + a.KT, __ldg(a.kend + U));
    const int sa = __ldg(a.bra.shA + P), sb = __ldg(a.bra.shB + P);
    const int oa = __ldg(a.ao + sa), ob = __ldg(a.ao + sb);
    const double QP = __ldg(a.bra.Q + P);
    for (int i = lane; i < C::NAB; i += 32) jab[i] = 0.0;
    __syncwarp();
    for (int R = r0; R < r1; ++R) {
      const double QQ = QP * __ldg(a.ket.Q + R);
      if (QQ < a.thresh) continue;
      const int sc = __ldg(a.ket.shA + R), sd = __ldg(a.ket.shB + R);
      if (!dw_keep<DW>(a, QQ, sa, sb, sc, sd)) continue;
      const int oc = __ldg(a.ao + sc), od = __ldg(a.ao + sd);
      d_prefetch<C>(jab + C::NAB, a.D, oa, ob, oc, od, a.nbf, lane);
      quartet_block<C>(a.bra, P, a.ket, R, Rbuf, V, htab, rtab, a.boys, lane);
      double deg = 1.0;
      if (sa == sb) deg *= 0.5;
      if (sc == sd) deg *= 0.5;
      if (a.same_bucket && P == R) deg *= 0.5;
      digest<C, false>(V, deg, oa, ob, oc, od, a.D, a.nbf, a.J, a.K, jab, jab + C::NAB, Rbuf, lane);
      __syncwarp();
    }
    for (int ab = lane; ab < C::NAB; ab += 32)
      {  // J_ab block, oriented for contiguous runs (blk_rc, eri_core.cuh)
        int i, j;
        blk_rc<C::NA, C::NB>(ab, i, j);
        atomicAdd(a.J + blk_dst<C::NA, C::NB>(oa + i, ob + j, a.nbf), jab[i * C::NB + j]);
      }
    __syncwarp();
  }
  }
}

// eri_batch store epilogue: canonical V[A][B][C][D] -> user order [a][b][c][d] (undo the swaps)
template <class C>
__device__ void store_block(const BatchArgs& a, int qi, const double* __restrict__ V, int lane) {
  const int fl = a.qflag[qi];
  const bool sab = fl & 1, scd = fl & 2, sbk = fl & 4;
  const int n[4] = {C::NA, C::NB, C::NC, C::ND};
  // user positions of the canonical shells A, B, C, D, and the sizes in user order
  const int posA = sbk ? (scd ? 3 : 2) : (sab ? 1 : 0);
  const int posB = sbk ? (scd ? 2 : 3) : (sab ? 0 : 1);
  const int posC = sbk ? (sab ? 1 : 0) : (scd ? 3 : 2);
  const int posD = sbk ? (sab ? 0 : 1) : (scd ? 2 : 3);
  int nu[4];
  nu[posA] = n[0]; nu[posB] = n[1]; nu[posC] = n[2]; nu[posD] = n[3];
  const size_t base = (size_t)a.qout[qi];
  for (int e = lane; e < C::NAB * C::NCD; e += 32) {
    int idx[4];
    const int ab = e / C::NCD, cd = e % C::NCD;
    idx[posA] = ab / C::NB; idx[posB] = ab % C::NB; idx[posC] = cd / C::ND; idx[posD] = cd % C::ND;
    a.out[base + (((size_t)idx[0] * nu[1] + idx[1]) * nu[2] + idx[2]) * nu[3] + idx[3]] = V[e];
  }
}

// Reduced-precision tier of the persistent J/K kernel (eri_quant.cuh): the task loop and the FP64
// digestion of jk_body, the TF32 basis transformation of quartet_block_q.
template <class C>
__host__ __device__ constexpr int q_warps() { return warps_for<C, ClsQ<C>::WARP_DBL>(); }
template <class C>
__host__ __device__ constexpr size_t cta_smem_bytes_q() {
  return (size_t)C::HTAB_BYTES + C::RTAB_BYTES + sizeof(double) * (size_t)q_warps<C>() * ClsQ<C>::WARP_DBL;
}
template <int X, int Y, bool DW = false>
__global__ void __launch_bounds__(CTA_THREADS) jk_kernel_q(JKArgs a) {
  using C = ClsXY<X, Y>;
  using Q = ClsQ<C>;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  uint16_t* htab = reinterpret_cast<uint16_t*>(smem_raw);
  uint32_t* rtab = reinterpret_cast<uint32_t*>(smem_raw + C::HTAB_BYTES);
  double* wbase = reinterpret_cast<double*>(smem_raw + C::HTAB_BYTES + C::RTAB_BYTES);
  init_tables<C>(htab, rtab);
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  double* Rbuf = wbase + (size_t)warp * Q::WARP_DBL;
  double* V = Rbuf + C::W_R;
  double* jab = V + C::W_V;
  float* R32 = reinterpret_cast<float*>(Rbuf + C::WARP_DBL);
  for (;;) {
  long long tg0, tg1;
  if (!grab_tasks(a, lane, tg0, tg1)) break;
  int U = find_entry(a, tg0);
  for (long long task = tg0; task < tg1; ++task) {
    while (__ldg(a.task_off + U + 1) <= task) ++U;
    const int P = __ldg(a.ent_P + U);
    const int r0 = __ldg(a.kbeg + U) + (int)(task - __ldg(a.task_off + U)) * a.KT;
    const int r1 = min(r0 + a.KT, __ldg(a.kend + U));
    const int sa = __ldg(a.bra.shA + P), sb = __ldg(a.bra.shB + P);
    const int oa = __ldg(a.ao + sa), ob = __ldg(a.ao + sb);
    const double QP = __ldg(a.bra.Q + P);
    for (int i = lane; i < C::NAB; i += 32) jab[i] = 0.0;
    __syncwarp();
    for (int R = r0; R < r1; ++R) {
      const double QQ = QP * __ldg(a.ket.Q + R);
      if (QQ < a.thresh) continue;
      const int sc = __ldg(a.ket.shA + R), sd = __ldg(a.ket.shB + R);
      if (!dw_keep<DW>(a, QQ, sa, sb, sc, sd)) continue;
      const int oc = __ldg(a.ao + sc), od = __ldg(a.ao + sd);
      d_prefetch<C>(jab + C::NAB, a.D, oa, ob, oc, od, a.nbf, lane);
      quartet_block_q<C>(a.bra, P, a.ket, R, Rbuf, R32, V, htab, rtab, a.boys, lane);
      double deg = 1.0;
      if (sa == sb) deg *= 0.5;
      if (sc == sd) deg *= 0.5;
      if (a.same_bucket && P == R) deg *= 0.5;
      digest<C, false>(V, deg, oa, ob, oc, od, a.D, a.nbf, a.J, a.K, jab, jab + C::NAB, Rbuf, lane);
      __syncwarp();
    }
    for (int ab = lane; ab < C::NAB; ab += 32)
      {  // J_ab block, oriented for contiguous runs (blk_rc, eri_core.cuh)
        int i, j;
        blk_rc<C::NA, C::NB>(ab, i, j);
        atomicAdd(a.J + blk_dst<C::NA, C::NB>(oa + i, ob + j, a.nbf), jab[i * C::NB + j]);
      }
    __syncwarp();
  }
  }
}

// TF32-tier batch kernel (store epilogue only): eri_batch with MAKO_ERI_REDUCED
template <int X, int Y>
__global__ void __launch_bounds__(CTA_THREADS) batch_kernel_q(BatchArgs a) {
  using C = ClsXY<X, Y>;
  using Q = ClsQ<C>;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  uint16_t* htab = reinterpret_cast<uint16_t*>(smem_raw);
  uint32_t* rtab = reinterpret_cast<uint32_t*>(smem_raw + C::HTAB_BYTES);
  double* wbase = reinterpret_cast<double*>(smem_raw + C::HTAB_BYTES + C::RTAB_BYTES);
  init_tables<C>(htab, rtab);
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  double* Rbuf = wbase + (size_t)warp * Q::WARP_DBL;
  double* V = Rbuf + C::W_R;
  float* R32 = reinterpret_cast<float*>(Rbuf + C::WARP_DBL);
  for (int qi = blockIdx.x * (blockDim.x >> 5) + warp; qi < a.nq; qi += gridDim.x * (blockDim.x >> 5)) {
    quartet_block_q<C>(a.bra, a.qbra[qi], a.ket, a.qket[qi], Rbuf, R32, V, htab, rtab, a.boys, lane);
    store_block<C>(a, qi, V, lane);
    __syncwarp();
  }
}

// Batch kernel: one warp per listed quartet; store (eri_batch) or Schwarz-diagonal epilogue.
template <int X, int Y>
__global__ void __launch_bounds__(CTA_THREADS) batch_kernel(BatchArgs a) {
  using C = ClsXY<X, Y>;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  uint16_t* htab = reinterpret_cast<uint16_t*>(smem_raw);
  uint32_t* rtab = reinterpret_cast<uint32_t*>(smem_raw + C::HTAB_BYTES);
  double* wbase = reinterpret_cast<double*>(smem_raw + C::HTAB_BYTES + C::RTAB_BYTES);
  init_tables<C>(htab, rtab);
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  double* Rbuf = wbase + (size_t)warp * C::WARP_DBL;
  double* V = Rbuf + C::W_R;
  for (int qi = blockIdx.x * (blockDim.x >> 5) + warp; qi < a.nq; qi += gridDim.x * (blockDim.x >> 5)) {
    const int P = a.qbra[qi], R = a.qket[qi];
    quartet_block<C>(a.bra, P, a.ket, R, Rbuf, V, htab, rtab, a.boys, lane);
    if (a.diag) {
      double m = 0.0;
      for (int ab = lane; ab < C::NAB; ab += 32) m = fmax(m, fabs(V[ab * C::NCD + ab]));
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) m = fmax(m, __shfl_xor_sync(0xffffffffu, m, o));
      if (lane == 0) a.out[a.qout[qi]] = sqrt(m);
    } else {
      store_block<C>(a, qi, V, lane);
    }
    __syncwarp();
  }
}

template <int X, int Y>
static mako_status set_smem_attr(const void* fn, size_t smem) {
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return fail(MAKO_ERR_CUDA, std::string("cudaFuncSetAttribute: ") + cudaGetErrorString(e));
  return MAKO_OK;
}

template <int X, int Y>
int jk_blocks_per_sm() {
  using C = ClsXY<X, Y>;
  constexpr size_t smem = cta_smem_bytes<C>();
  static int cached = -1;
  if (cached < 0) {
    int nb = 0;
    if constexpr (use_kf_swap<X, Y>()) {
      constexpr size_t ks = KfCfg<Y, X>::SMEM;
      if (set_smem_attr<X, Y>((const void*)kf_jk_kernel_ptr<Y, X>(), ks)) return 1;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kf_jk_kernel_ptr<Y, X>(), CTA_THREADS, ks);
    } else if constexpr (use_kf<X, Y>()) {
      constexpr size_t ks = KfCfg<X, Y>::SMEM;
      if (set_smem_attr<X, Y>((const void*)kf_jk_kernel_ptr<X, Y>(), ks)) return 1;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kf_jk_kernel_ptr<X, Y>(), CTA_THREADS, ks);
    } else if constexpr (use_tpq(X, Y)) {
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, tpq_jk_kernel_ptr<X, Y>(), CTA_THREADS, 0);
    } else if constexpr (use_slab<X, Y>()) {
      constexpr size_t ss = SlabCfg<X, Y>::SMEM;
      if (set_smem_attr<X, Y>((const void*)slab_jk_kernel<X, Y>, ss)) return 1;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, slab_jk_kernel<X, Y>, CTA_THREADS, ss);
    } else if constexpr (use_jk_swap<X, Y>()) {
      using CS = ClsXY<Y, X>;
      constexpr size_t sms = cta_smem_bytes<CS>();
      if (set_smem_attr<X, Y>((const void*)jk_kernel_ptr<Y, X>(), sms)) return 1;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, jk_kernel_ptr<Y, X>(), 32 * jk_warps<CS>(), sms);
    } else {
      if (set_smem_attr<X, Y>((const void*)jk_kernel_ptr<X, Y>(), smem)) return 1;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, jk_kernel_ptr<X, Y>(), 32 * jk_warps<C>(), smem);
    }
    cached = nb < 1 ? 1 : nb;
  }
  return cached;
}

template <int X, int Y>
mako_status launch_jk_xy(const JKArgs& a, void* stream, int* nlaunch) {
  using C = ClsXY<X, Y>;
  constexpr size_t smem = cta_smem_bytes<C>();
  const long long ntask = a.ntask_local;
  if (ntask <= 0) return MAKO_OK;
  int dev = 0, nsm = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  const int bps = jk_blocks_per_sm<X, Y>();
  constexpr int WPC = (use_kf_swap<X, Y>() || use_kf<X, Y>() || use_tpq(X, Y) || use_slab<X, Y>()) ? CTA_WARPS
                                                                                                 : jk_warps<JkCls<X, Y>>();
  long long want = (ntask + WPC - 1) / WPC;
  long long cap = (long long)nsm * bps / (a.grid_div > 1 ? a.grid_div : 1);
  if (cap < nsm) cap = nsm;
  const int grid = (int)(want < cap ? want : cap);
  // density-weighted screening (a.dsh != null) runs separate instantiations, so the plain build's
  // kernels carry none of its code (it raised their register counts)
  const cudaStream_t cs = (cudaStream_t)stream;
  if constexpr (has_lowp<X, Y>()) {
    if (a.lowp) {
      constexpr int XQ = use_jk_swap<X, Y>() ? Y : X, YQ = use_jk_swap<X, Y>() ? X : Y;
      using CQ = ClsXY<XQ, YQ>;
      constexpr size_t sq = cta_smem_bytes_q<CQ>();
      // the TF32 tier's own occupancy (its SMEM is larger by the TF32 R rows)
      static int bq = -1;
      if (bq < 0) {
        if (set_smem_attr<X, Y>((const void*)jk_kernel_q<XQ, YQ>, sq) ||
            set_smem_attr<X, Y>((const void*)jk_kernel_q<XQ, YQ, true>, sq))
          return MAKO_ERR_CUDA;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bq, jk_kernel_q<XQ, YQ>, 32 * q_warps<CQ>(), sq);
        if (bq < 1) bq = 1;
      }
      constexpr int QW = q_warps<CQ>();
      const long long gq = std::min<long long>((ntask + QW - 1) / QW, std::max<long long>((long long)nsm * bq, nsm));
      if (a.dsh) jk_kernel_q<XQ, YQ, true><<<(int)gq, 32 * QW, sq, cs>>>(a);
      else jk_kernel_q<XQ, YQ><<<(int)gq, 32 * QW, sq, cs>>>(a);
      cudaError_t e = cudaGetLastError();
      if (e != cudaSuccess) return fail(MAKO_ERR_CUDA, std::string("jk_kernel_q launch: ") + cudaGetErrorString(e));
      if (nlaunch) ++*nlaunch;
      return MAKO_OK;
    }
  }
  if constexpr (use_kf_swap<X, Y>()) {
    if (a.dsh) {
      if (set_smem_attr<X, Y>((const void*)kf_jk_kernel_ptr<Y, X, true>(), KfCfg<Y, X>::SMEM)) return MAKO_ERR_CUDA;
      kf_jk_kernel_ptr<Y, X, true>()<<<grid, CTA_THREADS, KfCfg<Y, X>::SMEM, cs>>>(a);
    } else {
      kf_jk_kernel_ptr<Y, X>()<<<grid, CTA_THREADS, KfCfg<Y, X>::SMEM, cs>>>(a);
    }
  } else if constexpr (use_kf<X, Y>()) {
    if (a.dsh) {
      if (set_smem_attr<X, Y>((const void*)kf_jk_kernel_ptr<X, Y, true>(), KfCfg<X, Y>::SMEM)) return MAKO_ERR_CUDA;
      kf_jk_kernel_ptr<X, Y, true>()<<<grid, CTA_THREADS, KfCfg<X, Y>::SMEM, cs>>>(a);
    } else {
      kf_jk_kernel_ptr<X, Y>()<<<grid, CTA_THREADS, KfCfg<X, Y>::SMEM, cs>>>(a);
    }
  } else if constexpr (use_tpq(X, Y)) {
    // strip digestion (eri_tpq.cuh) is an experiment, off by default: it cuts the global FP64 atomics
    // of these classes 5.5x but moves the bound to the shared-memory CAS loops and costs occupancy
    // (measured 12.32 -> 13.12 s per build, S6); MAKO_STRIP=1 enables it where the strip fits
    static const bool strip = std::getenv("MAKO_STRIP") != nullptr;
    const size_t ss = tpq_strip_smem<X, Y>(a.nbf, a.nshell);
    if (strip && a.unit_off && ss <= SMEM_CTA_MAX) {
      const void* fn = a.dsh ? (const void*)tpq_strip_kernel<X, Y, true> : (const void*)tpq_strip_kernel<X, Y>;
      if (set_smem_attr<X, Y>(fn, ss)) return MAKO_ERR_CUDA;
      int nb = 0;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, tpq_strip_kernel<X, Y>, 32 * TPQ_STRIP_WARPS, ss);
      const long long gs = std::min<long long>((long long)nsm * std::max(nb, 1), a.nunit);
      if (a.dsh) tpq_strip_kernel<X, Y, true><<<(int)std::max<long long>(gs, 1), 32 * TPQ_STRIP_WARPS, ss, cs>>>(a);
      else tpq_strip_kernel<X, Y><<<(int)std::max<long long>(gs, 1), 32 * TPQ_STRIP_WARPS, ss, cs>>>(a);
    } else {
      if (a.dsh) tpq_jk_kernel_ptr<X, Y, true>()<<<grid, CTA_THREADS, 0, cs>>>(a);
      else tpq_jk_kernel_ptr<X, Y>()<<<grid, CTA_THREADS, 0, cs>>>(a);
    }
  } else if constexpr (use_slab<X, Y>()) {
    if (a.dsh) {
      if (set_smem_attr<X, Y>((const void*)slab_jk_kernel<X, Y, true>, SlabCfg<X, Y>::SMEM)) return MAKO_ERR_CUDA;
      slab_jk_kernel<X, Y, true><<<grid, CTA_THREADS, SlabCfg<X, Y>::SMEM, cs>>>(a);
    } else {
      slab_jk_kernel<X, Y><<<grid, CTA_THREADS, SlabCfg<X, Y>::SMEM, cs>>>(a);
    }
  } else if constexpr (use_jk_swap<X, Y>()) {
    constexpr size_t sms = cta_smem_bytes<ClsXY<Y, X>>();
    if (a.dsh) {
      if (set_smem_attr<X, Y>((const void*)jk_kernel_ptr<Y, X, true>(), sms)) return MAKO_ERR_CUDA;
      jk_kernel_ptr<Y, X, true>()<<<grid, 32 * WPC, sms, cs>>>(a);
    } else {
      jk_kernel_ptr<Y, X>()<<<grid, 32 * WPC, sms, cs>>>(a);
    }
  } else {
    if (a.dsh) {
      if (set_smem_attr<X, Y>((const void*)jk_kernel_ptr<X, Y, true>(), smem)) return MAKO_ERR_CUDA;
      jk_kernel_ptr<X, Y, true>()<<<grid, 32 * WPC, smem, cs>>>(a);
    } else {
      jk_kernel_ptr<X, Y>()<<<grid, 32 * WPC, smem, cs>>>(a);
    }
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(MAKO_ERR_CUDA, std::string("jk_kernel launch: ") + cudaGetErrorString(e));
  if (nlaunch) ++*nlaunch;
  return MAKO_OK;
}

template <int X, int Y>
mako_status launch_batch_xy(const BatchArgs& a, void* stream) {
  using C = ClsXY<X, Y>;
  constexpr size_t smem = cta_smem_bytes<C>();
  if (a.nq <= 0) return MAKO_OK;
  int grid = (a.nq + jk_warps<C>() - 1) / jk_warps<C>();
  if (grid > 148 * 64) grid = 148 * 64;
  if constexpr (has_lowp<X, Y>()) {
    if (a.lowp && !a.diag) {
      constexpr size_t sq = cta_smem_bytes_q<C>();
      mako_status st = set_smem_attr<X, Y>((const void*)batch_kernel_q<X, Y>, sq);
      if (st) return st;
      batch_kernel_q<X, Y><<<(a.nq + q_warps<C>() - 1) / q_warps<C>() < grid ? (a.nq + q_warps<C>() - 1) / q_warps<C>() : grid,
                             32 * q_warps<C>(), sq, (cudaStream_t)stream>>>(a);
      cudaError_t e = cudaGetLastError();
      if (e != cudaSuccess) return fail(MAKO_ERR_CUDA, std::string("batch_kernel_q launch: ") + cudaGetErrorString(e));
      return MAKO_OK;
    }
  }
  mako_status st = set_smem_attr<X, Y>((const void*)batch_kernel<X, Y>, smem);
  if (st) return st;
  batch_kernel<X, Y><<<grid, 32 * jk_warps<C>(), smem, (cudaStream_t)stream>>>(a);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(MAKO_ERR_CUDA, std::string("batch_kernel launch: ") + cudaGetErrorString(e));
  return MAKO_OK;
}

}  // namespace mako

namespace mako {
template <int X, int Y>
int task_kets_xy() {
  if constexpr (use_kf_swap<X, Y>()) return KfCfg<Y, X>::NK;
  else if constexpr (use_kf<X, Y>()) return KfCfg<X, Y>::NK;
  else if constexpr (use_tpq(X, Y)) return 32;
  else return 16;
}
template <int X, int Y>
bool swap_xy() {
  return use_kf_swap<X, Y>() || use_jk_swap<X, Y>();
}
template <int X, int Y>
bool lowp_xy() {
  return has_lowp<X, Y>();
}
}  // namespace mako

#define MAKO_INSTANTIATE(X, Y)                                                                   \
  template mako_status mako::launch_jk_xy<X, Y>(const mako::JKArgs&, void*, int*);               \
  template mako_status mako::launch_batch_xy<X, Y>(const mako::BatchArgs&, void*);               \
  template int mako::jk_blocks_per_sm<X, Y>();                                                   \
  template int mako::task_kets_xy<X, Y>();                                                       \
  template bool mako::swap_xy<X, Y>();                                                            \
  template bool mako::lowp_xy<X, Y>();
#endif
