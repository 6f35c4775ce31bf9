// mako_internal.h -- shared internal definitions of libmako (product path only).
//
// Hermite / Cartesian index conventions, class geometry, device-side data views.
// Nothing here is shared with oracle/ (the oracle is an independent implementation).
#pragma once

#include <cstdint>
#include <cstddef>
#include <string>
#include <vector>

#include "../../include/mako.h"

#ifdef __CUDACC__
#define MK_HD __host__ __device__
#else
#define MK_HD
#endif

namespace mako {

constexpr int LMAX = MAKO_LMAX;
constexpr int NBUCKET = (LMAX + 1) * (LMAX + 2) / 2;  // (la >= lb) pair buckets: ss ps pp ds dp dd fs fp fd ff gs gp gd gf gg
constexpr int NCLASS = NBUCKET * (NBUCKET + 1) / 2;

// number of Hermite (or Cartesian) tuples (t,u,v) with t+u+v <= L
MK_HD constexpr int nH(int L) { return L < 0 ? 0 : (L + 1) * (L + 2) * (L + 3) / 6; }
MK_HD constexpr int ncart(int l) { return (l + 1) * (l + 2) / 2; }
MK_HD constexpr int nsph(int l) { return 2 * l + 1; }
// Hermite index: degree-major, then t descending, then u descending.
MK_HD constexpr int hidx(int t, int u, int v) {
  return nH(t + u + v - 1) + (u + v) * (u + v + 1) / 2 + v;
}
// Cartesian index within a shell of degree l (lx descending, then ly descending): xx xy xz yy yz zz
MK_HD constexpr int cart_index(int x, int y, int z) { return (y + z) * (y + z + 1) / 2 + z; }
// pair bucket of (la >= lb)
MK_HD constexpr int bucket_of(int la, int lb) { return la * (la + 1) / 2 + lb; }

// Boys table: Taylor grid, F_m(T_k) for T_k = k * BOYS_H, k = 0..BOYS_NGRID-1, m = 0..BOYS_MMAX
constexpr double BOYS_H = 1.0 / 32.0;
constexpr double BOYS_TMAX = 40.0;
constexpr int BOYS_NGRID = 1281;      // T_k up to 40
constexpr int BOYS_MMAX = 24;         // supports L + 6 <= 24
constexpr int BOYS_NM = BOYS_MMAX + 1;
constexpr int BOYS_TAYLOR = 7;        // Taylor terms (|dT| <= 1/64 -> truncation < 5e-17 relative)
// per-L packed rows: block L (0 <= L < BOYS_LTAB), row k = {F_L..F_{L+6}(T_k), exp(-T_k)}: 64 B,
// read with four 128-bit loads (one cache line per lane and lookup)
constexpr int BOYS_LTAB = BOYS_MMAX - BOYS_TAYLOR + 2;  // L = 0..18
constexpr int BOYS_ROW = 8;
constexpr double BOYS_TEXP = 80.0;    // for 40 <= T < 80 exp(-T) comes from a second grid; beyond, it is
                                      // below 1e-18 of every F_m (m <= 12) and is dropped (reading R1)
constexpr int BOYS_NEXP = 1281;       // exp(-(40 + k/32)), k = 0..1280
constexpr size_t BOYS_EXP_OFF = (size_t)BOYS_LTAB * BOYS_NGRID * BOYS_ROW;
constexpr size_t BOYS_TABLE_DOUBLES = BOYS_EXP_OFF + BOYS_NEXP;

// Kernel family per class (X >= Y buckets).  Low-l classes use the lane-per-ket register kernel
// ("TPQ": Boys, R, contraction and digestion in registers of one lane), the rest the warp-per-quartet
// DMMA kernel.  Register estimate (doubles): R + V + W + cached ket E~ + cached bra E~.
MK_HD constexpr int b_la(int b) {  // bucket b = la (la + 1) / 2 + lb
  int la = 0;
  while ((la + 1) * (la + 2) / 2 <= b) ++la;
  return la;
}
MK_HD constexpr int b_lb(int b) { return b - b_la(b) * (b_la(b) + 1) / 2; }
MK_HD constexpr int tpq_regs(int X, int Y) {
  return nH(b_la(X) + b_lb(X) + b_la(Y) + b_lb(Y)) + nsph(b_la(X)) * nsph(b_lb(X)) * nsph(b_la(Y)) * nsph(b_lb(Y)) +
         nsph(b_la(Y)) * nsph(b_lb(Y)) * (1 + nH(b_la(Y) + b_lb(Y))) +
         (nsph(b_la(X)) * nsph(b_lb(X)) * nH(b_la(X) + b_lb(X)) <= 40 ? nsph(b_la(X)) * nsph(b_lb(X)) * nH(b_la(X) + b_lb(X)) : 0);
}
MK_HD constexpr bool use_tpq(int X, int Y) { return Y <= 1 && b_la(X) <= 3 && tpq_regs(X, Y) <= 100; }
MK_HD constexpr int class_kt(int X, int Y) { return use_tpq(X, Y) ? 32 : 16; }

// reduced-precision tier: floats per primitive pair of the TF32 fragment-order copies of E~ (pairs.cu
// build_lowp_kernel, read by eri_quant.cuh): GEMM1 A fragments (m16 x k8 tiles) and GEMM2 B fragments
// (k8 x n8 tiles)
MK_HD constexpr int lowp_a_floats(int la, int lb) {
  return ((nsph(la) * nsph(lb) + 15) / 16) * ((nH(la + lb) + 7) / 8) * 128;
}
// FP64 fragment-order copies (m8n8k4): doubles per primitive pair
MK_HD constexpr int frag_a_doubles(int la, int lb) { return ((nsph(la) * nsph(lb) + 7) / 8) * ((nH(la + lb) + 3) / 4) * 32; }
MK_HD constexpr int frag_b_doubles(int la, int lb) { return ((nH(la + lb) + 7) / 8) * ((nsph(la) * nsph(lb) + 7) / 8) * 64; }
MK_HD constexpr int lowp_b_floats(int la, int lb) {
  return ((nH(la + lb) + 7) / 8) * ((nsph(la) * nsph(lb) + 7) / 8) * 64;
}

// Pair buckets are ordered by (primitive-pair count group, Q descending): inside a group the
// Schwarz-surviving kets of a bra are still a prefix, and the kets of one warp task share a similar
// K_CD (uniform per-lane primitive loops).  Groups: K = 1, 2, 3, 4, 5-6, 7-9, 10-12, 13-16, 17-24,
// 25-36, 37+.
constexpr int NKGROUP = 11;
MK_HD constexpr int kgroup(int K) {
  return K <= 4 ? (K < 1 ? 0 : K - 1)
                : (K <= 6 ? 4 : (K <= 9 ? 5 : (K <= 12 ? 6 : (K <= 16 ? 7 : (K <= 24 ? 8 : (K <= 36 ? 9 : 10))))));
}

// Per-class kernel-family choices, measured on the bench workload (profiles/README.md; re-selected in round 2
// from all-on / all-off runs per family, profiles/bench_r02_ab.md: (dp|ps) left the ket-first kernel for the
// lane-per-ket one, 531 -> 482 ms; (ff|dd) and (ff|fd) run transposed).  Codes are X * 100 + Y.  Overridable
// with -D for experiment builds (build.py --variant).
#ifndef MAKO_KF_PICK
#define MAKO_KF_PICK 303, 403, 501, 603, 701, 800, 801, 900, 700, 500
#endif
#ifndef MAKO_KFSWAP_PICK
#define MAKO_KFSWAP_PICK 302
#endif
// warp-per-quartet classes run transposed ((ab|cd) as (cd|ab): the ket side takes the inner, per
// primitive-quartet GEMM1; S6), measured per class
#ifndef MAKO_JKSWAP_PICK
#define MAKO_JKSWAP_PICK 703, 803, 706, 503, 802, 806, 901, 804, 502, 807, 504, 906, 903, 907, 702, 904, 805, 902, 905, 908
#endif
#ifndef MAKO_SLAB_PICK
#define MAKO_SLAB_PICK 402
#endif
#ifndef MAKO_JK_CAP4
#define MAKO_JK_CAP4 800, 801, 802, 803, 804, 805, 806, 807, 705, 408, 209, 609
#endif
#ifndef MAKO_KF_CAP3
#define MAKO_KF_CAP3 203, 701, 800, 303, 900, 501
#endif
constexpr int kKfPick[] = {MAKO_KF_PICK};
constexpr int kKfSwapPick[] = {MAKO_KFSWAP_PICK};
constexpr int kSlabPick[] = {MAKO_SLAB_PICK};
constexpr int kJkSwapPick[] = {MAKO_JKSWAP_PICK};
// warp-per-quartet classes (codes bucket(la,lb) * 100 + bucket(lc,ld) of the evaluated orientation)
// whose contracted quartets take the batched lane-per-quartet R path (eri_core.cuh quartet_block_rb)
#ifndef MAKO_RBATCH_PICK
#define MAKO_RBATCH_PICK 207, 205, 602, 404, 202, 307
#endif
constexpr int kRBatchPick[] = {MAKO_RBATCH_PICK};
// warp-per-quartet classes (same codes) whose GEMM2 B operands are read from the row-major E~ rather
// than the fragment-order copy (measured per class, profiles/bench_r02_ab.md)
#ifndef MAKO_NOFRAGB_PICK
#define MAKO_NOFRAGB_PICK 707, 602, 207, 109, 705, 309, 808, 205, 908, 905
#endif
constexpr int kNoFragBPick[] = {MAKO_NOFRAGB_PICK};
constexpr int kJkCap4[] = {MAKO_JK_CAP4};
constexpr int kKfCap3[] = {MAKO_KF_CAP3};
template <int N>
MK_HD constexpr bool in_list(const int (&a)[N], int v) {
  for (int i = 0; i < N; ++i)
    if (a[i] == v) return true;
  return false;
}

// task -> entry lookup: every TASK_SAMPLE-th task's entry is stored, the rest is a short forward scan
constexpr int TASK_SAMPLE_SHIFT = 4;
constexpr int TASK_SAMPLE = 1 << TASK_SAMPLE_SHIFT;

#ifndef MAKO_TASK_GRAB
#define MAKO_TASK_GRAB 4
#endif
constexpr int TASK_GRAB = MAKO_TASK_GRAB;  // tasks taken per counter increment (one entry lookup per grab)

// Interleaved shard split: the task index space [0, T) of a class is cut into chunks of
// C tasks (C a multiple of TASK_GRAB, about 256 chunks per shard); shard s owns chunks j = s, s + n,
// s + 2n, ...  A pure function of (T, n): every rank derives the same split.
MK_HD inline long long shard_chunk(long long T, int n) {
  long long c = T / ((long long)n * 256);
  c = (c + TASK_GRAB - 1) / TASK_GRAB * TASK_GRAB;
  return c < 4 * TASK_GRAB ? 4 * TASK_GRAB : c;
}
// number of tasks of shard s
MK_HD inline long long shard_ntask(long long T, int s, int n, long long C) {
  const long long nch = (T + C - 1) / C;  // chunks, the last one possibly partial
  if (s >= nch) return 0;
  const long long mine = (nch - 1 - s) / n + 1;  // chunks s, s+n, ... < nch
  const long long last = s + (mine - 1) * n;
  return (mine - 1) * C + ((last == nch - 1) ? T - last * C : C);
}
// global task of local task index l of shard s
MK_HD inline long long shard_task(long long l, int s, int n, long long C) {
  return ((l / C) * n + s) * C + l % C;
}

// primitive-pair screening (reading R7)
constexpr double PRIM_PAIR_EPS = 1e-18;

// ---------------------------------------------------------------------------
// Device view of one bucket of a pair set (all device pointers)
// ---------------------------------------------------------------------------
struct PairView {
  int n;                 // pairs in the bucket
  int la, lb;
  const int* shA;        // [n] shell with the higher l (la >= lb)
  const int* shB;        // [n]
  const double* Q;       // [n] Schwarz factors (may be null during Schwarz computation)
  const int* poff;       // [n+1] primitive-pair offsets
  const double* pdat;    // [nprim][4]: p, Px, Py, Pz
  const double* Ebra;    // [nprim][nab][nHab]  E~ with spherical transform, coefficients, 1/p folded
  const double* Eket;    // [nprim][nHab][nab]  (-1)^{|q|} E~^T
  // FP64 copies in mma.m8n8k4 fragment order (one coalesced warp load per fragment; pairs.cu
  // build_frag_kernel): GEMM1 A fragments [nprim][MT8][KS4][32 lanes] of E~ and GEMM2 B fragments
  // [nprim][NT8(q)][NT8(cd)][32 lanes][2] of (-1)^{|q|} E~^T
  const double* EbraD;
  const double* EketD;
  // reduced-precision tier (null until first requested): TF32 copies in mma fragment order
  const float* EbraF;    // [nprim][MT16][KS8][32 lanes][4]  GEMM1 A fragments of E~
  const float* EketF;    // [nprim][NT8(q)][NT8(cd)][32 lanes][2]  GEMM2 B fragments of (-1)^{|q|} E~^T
};

// arguments of a J/K class launch
struct JKArgs {
  PairView bra, ket;
  int same_bucket;
  // shard of the class's task index space [0, ntask): the tasks are cut into chunks of
  // `chunk` consecutive tasks, chunk j belongs to shard j mod nshards (interleaved, so every shard
  // samples the whole Q-sorted cost profile of the class); this launch walks its ntask_local tasks
  long long ntask, ntask_local, chunk;
  int shard, nshards;
  const long long* task_off;        // [nent+1] task prefix per non-empty (bra pair, ket K-group) entry
  const int* ent_P;                 // [nent] bra pair of the entry
  const int* kbeg;                  // [nent] first ket of the entry (start of its K-group segment)
  const int* kend;                  // [nent] one past the last surviving ket (Q-sorted prefix of the segment)
  const int* usamp;                 // [ntask / TASK_SAMPLE + 1] entry holding task k * TASK_SAMPLE
  int nent;
  // bra units (strip digestion, eri_tpq.cuh): unit u = tasks [unit_off[u], unit_off[u+1]) of bra pair unit_P[u]
  int nunit;
  const long long* unit_off;        // [nunit + 1]
  const int* unit_P;                // [nunit]
  const int* shl;                   // [nshell] angular momentum of every shell
  int KT;                           // kets per task
  unsigned long long* counter;      // dynamic task counter (zeroed before launch)
  const double* D;
  double* J;                        // accumulators (symmetrised afterwards)
  double* K;
  int nbf;
  const int* ao;                    // [nshell] AO offsets
  double thresh;
  // density-weighted screening (flag MAKO_JK_DENSITY_SCREEN; null = off): keep a quartet iff
  // Q_ab Q_cd max(|D| over its six shell blocks) >= dw_thresh; dsh[sa * nshell + sb] = max |D| of block
  const float* dsh;
  int nshell;
  double dw_thresh;
  const double* boys;               // Boys table
  int grid_div;                     // host side: grid = resident capacity / grid_div (concurrent classes)
  int lowp;                         // host side: run the class's TF32-tier kernel (eri_quant.cuh)
};

// arguments of a store/diag class launch (eri_batch, Schwarz)
struct BatchArgs {
  PairView bra, ket;
  int nq;
  const int* qbra;        // [nq] bra pair index in bucket
  const int* qket;        // [nq] ket pair index
  const long long* qout;  // [nq] output offset (store mode) or Q index (diag mode)
  const int* qflag;       // [nq] bit0 swap a/b, bit1 swap c/d, bit2 swap bra/ket (store mode)
  double* out;
  const double* boys;
  int diag;               // 1 = Schwarz mode: out[qout[i]] = sqrt(max |(ab|ab)|)
  int lowp;               // store mode: TF32-tier kernel where the class has one
};

}  // namespace mako
