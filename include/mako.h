/*
 * mako.h -- C ABI of the B200-native direct-SCF J/K library (libmako.so).
 *
 * The one data-parallel hot path of Mako (Han et al., "Matrix Is All You Need", SC'25;
 * PAPER.md = /root/reference/PAPER.md): electron-repulsion integrals evaluated as
 * matrix-shaped McMurchie-Davidson stages per angular-momentum class and contracted with a
 * density matrix into Coulomb and exchange matrices.
 *
 *   ERI       (ab|cd) = double integral phi_a(r1) phi_b(r1) |r1-r2|^-1 phi_c(r2) phi_d(r2)
 *                                                              PAPER.md:L106-L109 (S2.1, Eq. 1)
 *   basis     phi = sum_i c_i varphi_i (contracted Gaussians), shells of 2l+1 spherical functions
 *                                                              PAPER.md:L111-L119 (Eq. 2)
 *   MMD       [r]^(m) from the Boys seed, Eq. 5 recursion, [p|q] = (-1)^{l_q}[p+q]^(0),
 *             [ab|q] = sum_p E_ab^p [p|q], (ab|cd) = sum_q E_cd^q [ab|q]
 *                                                              PAPER.md:L164-L190 (Eq. 4-7), Alg. 1
 *   J/K       J_{mn} = sum_{ls} (mn|ls) D_{ls},  K_{ml} = sum_{ns} (mn|ls) D_{ns}
 *                                                              BASELINE.json north_star; FP64 Fock L296
 *   screening Schwarz Q_ab = sqrt(max_{m in a, n in b} |(mn|mn)|); a quartet is kept iff
 *             Q_ab * Q_cd >= thresh                             PAPER.md:L286, L300 (reading R6)
 *
 * Conventions (all functions):
 *   - Units: bohr, Hartree.  FP64 everywhere.
 *   - AO order: shells in input order; inside a shell, spherical functions p = (x, y, z) and for
 *     l >= 2 real solid harmonics m = -l..l with positive leading terms (PySCF-compatible).
 *     Only pure (spherical) functions are supported by the GPU path (pure = 1); pure = 0 returns
 *     MAKO_ERR_UNSUPPORTED.
 *   - Contraction coefficients refer to normalised primitives; the library renormalises each
 *     contracted shell so that its x^l Cartesian component has unit norm (pure functions then
 *     come out normalised).  Angular momentum l <= MAKO_LMAX.
 *   - Matrices (D, J, K) are dense nbf x nbf row-major FP64 in DEVICE memory, caller-owned
 *     (allocated e.g. by torch).  D must be symmetric.
 *   - Handles are library-owned: create/destroy pairs.  A handle is bound to the CUDA device that
 *     was current when it was created.
 *   - Asynchrony: functions taking a cuda_stream enqueue their device work on that stream
 *     (cudaStream_t passed as void*, NULL = legacy default stream) and return once it is enqueued;
 *     argument errors are reported immediately.
 *   - Errors: every function returns mako_status; on non-OK, mako_last_error() gives a
 *     thread-local message.  No exceptions escape, nothing is printed, nothing exits.
 *   - There is no CPU fallback: without a CUDA device every compute entry point returns
 *     MAKO_ERR_CUDA.
 */
#ifndef MAKO_H
#define MAKO_H

#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MAKO_LMAX 4

typedef enum {
  MAKO_OK = 0,
  MAKO_ERR_INVALID = 1,      /* NULL pointer, non-finite input, size mismatch, thresh < 0, bad shard */
  MAKO_ERR_UNSUPPORTED = 2,  /* l > MAKO_LMAX, pure == 0 */
  MAKO_ERR_CUDA = 3,         /* CUDA runtime error or no device */
  MAKO_ERR_OOM = 4,          /* device allocation failed */
  MAKO_ERR_STATE = 5         /* handle used on the wrong device / destroyed */
} mako_status;

typedef struct mako_basis_s* mako_basis;  /* opaque, library-owned */
typedef struct mako_pairs_s* mako_pairs;  /* opaque, library-owned, device-resident pair data */

/* Create a basis (Eq. 2).  All arrays are HOST pointers, copied.
 *   natm, Z[natm]            nuclear charges (only validated and stored; not used by ERIs)
 *   xyz[natm*3]              atom positions, bohr
 *   nshell                   number of shells
 *   shell_atom[nshell]       atom index of each shell (0 <= . < natm); the shell centre is xyz[atom]
 *   shell_l[nshell]          angular momentum 0..MAKO_LMAX
 *   shell_nprim[nshell]      primitives per shell (>= 1)
 *   exps[sum nprim]          primitive exponents (> 0), concatenated in shell order
 *   coefs[sum nprim]         contraction coefficients for normalised primitives, concatenated
 *   pure                     1 = spherical (2l+1) functions; 0 -> MAKO_ERR_UNSUPPORTED
 *   out                      receives the handle
 * Host-only: normalisation and the Cartesian->spherical tables; copies shell data to the device. */
mako_status mako_basis_create(int natm, const int* Z, const double* xyz, int nshell, const int* shell_atom,
                              const int* shell_l, const int* shell_nprim, const double* exps, const double* coefs,
                              int pure, mako_basis* out);
mako_status mako_basis_nbf(mako_basis basis, int* nbf);
mako_status mako_basis_nshell(mako_basis basis, int* nshell);
/* AO offset of every shell: ao_offset[nshell+1] (host), ao_offset[nshell] = nbf. */
mako_status mako_basis_ao_offsets(mako_basis basis, int* ao_offset);
void mako_basis_destroy(mako_basis basis);

/* Shell-pair data + Schwarz screening (Alg. 1 inputs
 * E_AB/E_CD, L286/L300 screening).  On the device: Hermite expansion matrices E~_ab (spherical
 * transform, contraction coefficients and 1/p folded in) for every primitive pair, the diagonal
 * ERIs (ab|ab) -> Q_ab.  Pairs with Q_ab * Q_max < thresh are dropped; survivors are bucketed by
 * (la, lb) and sorted by Q descending.  Primitive pairs with exp(-mu |AB|^2) < 1e-18 are dropped
 * (reading R7).  thresh >= 0 (0 keeps every pair).  Synchronises cuda_stream. */
mako_status mako_shellpairs_screen(mako_basis basis, double thresh, void* cuda_stream, mako_pairs* out);
/* counts: number of significant shell pairs, primitive pairs, and canonical shell quartets that
 * survive thresh (computed on the host from the sorted Q lists).  Any pointer may be NULL. */
mako_status mako_pairs_stats(mako_pairs pairs, double thresh, long long* n_pairs, long long* n_prim_pairs,
                             long long* n_quartets);
/* Algorithmic FP64 FLOPs of the two Hermite->AO contractions (Eq. 7) summed over
 * the canonical quartets of shard `shard` of `nshards` at thresh (unpadded spherical dims):
 *   sum_q [ K_AB K_CD 2 n_ab nH_ab nH_cd + K_CD 2 n_ab nH_cd n_cd ]  (DESIGN.md S "Measurement"). */
mako_status mako_pairs_flops(mako_pairs pairs, double thresh, int shard, int nshards, double* gemm_flops,
                             long long* n_quartets, long long* n_prim_quartets);
void mako_pairs_destroy(mako_pairs pairs);

/* Direct J/K build (the hot path; north_star).
 *   D     device nbf x nbf row-major FP64, symmetric, caller-owned (read only)
 *   J, K  device nbf x nbf row-major FP64, caller-owned, OVERWRITTEN (not accumulated) with
 *         J_{mn} = sum_{ls} (mn|ls) D_ls and K_{ml} = sum_{ns} (mn|ls) D_ns over the quartets of
 *         this shard that survive Q_ab Q_cd >= thresh.  Both come out exactly symmetric.
 *   thresh >= the pairs' screening threshold (smaller values are treated as equal to it).
 *   shard, nshards: 0 <= shard < nshards.  The canonical quartet tasks of every angular-momentum
 *         class (in bra-Q-descending order) are cut into chunks of C consecutive tasks (C a multiple
 *         of 4, about 256 chunks per shard); chunk j belongs to shard j mod nshards (interleaved, so
 *         every shard samples the whole cost profile of the class).
 *         A pure function of (pairs, thresh, shard, nshards): summing J/K over all shards gives the
 *         nshards = 1 result up to FP64 summation order.
 *   cuda_stream: all work is enqueued on it (async).  J, K, D must not alias.  Builds on one pairs
 *         handle are serialised: a build first waits (on cuda_stream) for the previous build of the
 *         same handle, whatever stream that one was enqueued on (the task counters, the D block maxima
 *         and the accumulate scratch are per-handle state). */
mako_status mako_build_jk(mako_pairs pairs, const double* D, double thresh, double* J, double* K, int shard,
                          int nshards, void* cuda_stream);

/* Density-weighted screening (S3.2.3 "density-weighted Schwarz ... pruned"; SURVEY
 * S8.f row 2; reading R17).  With flags = MAKO_JK_DENSITY_SCREEN, mako_build_jk_ex keeps a
 * canonical quartet only if, in addition to Q_ab Q_cd >= the pairs' threshold,
 *     Q_ab Q_cd Dmax(ab,cd) >= thresh,
 * Dmax(ab,cd) = the largest max|D_mn| over the six shell blocks (ab)(cd)(ac)(ad)(bc)(bd) the quartet
 * is contracted with.  A dropped quartet changes no J or K element by more than 2*thresh (its
 * |(mn|ls)| <= Q_ab Q_cd by Cauchy-Schwarz, and each of its J/K updates is (degeneracy <= 1) x 2 x
 * |(mn|ls) D|).  Intended for incremental SCF builds (D = Delta D).  This mode computes the block
 * maxima on the device and SYNCHRONISES cuda_stream once (the task plan depends on max|D|);
 * otherwise identical to mako_build_jk (flags = 0 is exactly mako_build_jk). */
#define MAKO_JK_DENSITY_SCREEN 1u
/* flags |= MAKO_JK_ACCUMULATE: J and K are ACCUMULATED (J += J[D], K += K[D]) instead of overwritten.
 * Used for incremental SCF builds on a density change (PAPER.md:L300 convergence-aware scheduling;
 * SURVEY S8.f row 2): J[D_n] = J[D_{n-1}] + J[D_n - D_{n-1}] (J, K linear in D).  The build's own
 * accumulators then live in a per-handle scratch of 2 nbf^2 doubles (allocated on first use), added
 * into J/K by the final symmetrisation kernel.  Valid for mako_build_jk_ex and mako_build_jk_mixed. */
#define MAKO_JK_ACCUMULATE 2u
mako_status mako_build_jk_ex(mako_pairs pairs, const double* D, double thresh, unsigned flags, double* J, double* K,
                             int shard, int nshards, void* cuda_stream);

/* Stage-aware reduced-precision J/K build (QuantMako, PAPER.md S3.2 L286-L302; SURVEY S8.f row 1;
 * DESIGN.md readings R19-R20).  Three tiers per canonical quartet ("critical ones are
 * evaluated with FP64 kernels, moderately important ones with quantized kernels, and negligible ones
 * are pruned"):
 *   Q_ab Q_cd < thresh (or the density rule of MAKO_JK_DENSITY_SCREEN)          pruned
 *   Q_ab Q_cd max|D| < T, T = thresh_fp64 / max|D| rounded DOWN to a power of 10,
 *     times max|D|  (i.e. a quartet whose J/K contribution bound is below ~thresh_fp64)
 *                                                                                 reduced precision
 *   otherwise                                                                      FP64
 * max|D| is the global maximum |D_mn|.  The reduced tier keeps the Boys function and the R recursion
 * in FP64, runs both Hermite->AO contractions (Eq. 7) as TF32 tensor-core GEMMs
 * with FP32 accumulation (L296 first stage) and digests into FP64 J/K (L296 second stage).  Classes
 * without a reduced-precision kernel (mako_class_reduced) run FP64 in both tiers.  Per-quartet error
 * budget: |d(ab|cd)| <= (2^-9 + (K1+K2) 2^-24) * sum|E~ R E~| (eri_quant.cuh).  thresh_fp64 > 0
 * (finite); thresh as in mako_build_jk_ex; flags: MAKO_JK_DENSITY_SCREEN and/or MAKO_JK_ACCUMULATE.  SYNCHRONISES
 * cuda_stream once (max|D| decides the tier plan).  D, J, K as in mako_build_jk. */
mako_status mako_build_jk_mixed(mako_pairs pairs, const double* D, double thresh, double thresh_fp64,
                                unsigned flags, double* J, double* K, int shard, int nshards, void* cuda_stream);
/* Density change of an incremental build: dD = D - D_prev (DEVICE nbf x nbf FP64,
 * caller-owned; dD must not alias D or D_prev) and *dmax = max |dD| (HOST), which the caller's
 * convergence-aware threshold schedule needs.  Enqueued on cuda_stream, then SYNCHRONISES it (dmax is
 * returned).  A non-finite entry returns MAKO_ERR_INVALID (after writing dD). */
mako_status mako_density_delta(mako_pairs pairs, const double* D, const double* D_prev, double* dD, double* dmax,
                               void* cuda_stream);
/* family[MAKO_NCLASS] (HOST): the kernel family that runs each class (S6): 0 lane-per-ket
 * register kernel, 1 ket-first DMMA kernel, 2 ket-first transposed, 3 slot-batched DMMA kernel,
 * 4 warp-per-quartet DMMA kernel, 5 warp-per-quartet transposed ((ab|cd) evaluated as (cd|ab)).
 * For measurement reports. */
mako_status mako_class_family(int* family);
/* mask[MAKO_NCLASS] (HOST): 1 where the class has a reduced-precision (TF32) kernel. */
mako_status mako_class_reduced(int* mask);

/* Number of CUDA kernels one mako_build_jk call launches for these arguments (for bench accounting). */
mako_status mako_build_jk_launches(mako_pairs pairs, double thresh, int shard, int nshards, int* n_launches);

/* Number of angular-momentum classes (bra bucket X >= ket bucket Y over the 15 (la>=lb) pair
 * buckets ss ps pp ds dp dd fs fp fd ff gs gp gd gf gg): class index c = X(X+1)/2 + Y. */
#define MAKO_NCLASS 120

/* Per-class algorithmic GEMM FLOPs (same definition as mako_pairs_flops) and quartet counts of
 * shard `shard`/`nshards` at thresh.  flops, quartets, prim_quartets: HOST arrays of MAKO_NCLASS (any NULL). */
mako_status mako_pairs_class_flops(mako_pairs pairs, double thresh, int shard, int nshards, double* flops,
                                   long long* quartets, long long* prim_quartets);

/* Measurement hooks.  mako_profile_enable(pairs, 1) resets and starts recording a CUDA event pair
 * around every class-kernel launch of subsequent mako_build_jk calls (on their stream);
 * mako_profile_read synchronises those events and returns, per class index, the summed kernel
 * milliseconds and the number of launches since enable (HOST arrays of MAKO_NCLASS, either NULL).
 * enable = 0 stops recording and frees the events. */
mako_status mako_profile_enable(mako_pairs pairs, int enable);
mako_status mako_profile_read(mako_pairs pairs, double* ms, long long* launches);

/* Test entry: nq shell quartets, quartets[4*q .. 4*q+3] = shell indices (a,b,c,d) in
 * any order (HOST array).  out (DEVICE, FP64) receives the blocks (ab|cd) concatenated in quartet
 * order, each laid out [n_a][n_b][n_c][n_d] in the AO order of each shell.  out_len (elements) must
 * equal the total size.  No screening.  Enqueued on cuda_stream; synchronises it before returning
 * (the temporary pair data is freed). */
mako_status mako_eri_batch(mako_basis basis, int nq, const int* quartets, double* out, size_t out_len,
                           void* cuda_stream);
/* As mako_eri_batch; flags = MAKO_ERI_REDUCED evaluates the quartets of classes that have a
 * reduced-precision kernel with it (the tier mako_build_jk_mixed uses; for its error budget and RMSE,
 * PAPER.md Table 2).  flags = 0 is exactly mako_eri_batch. */
#define MAKO_ERI_REDUCED 1u
mako_status mako_eri_batch_ex(mako_basis basis, int nq, const int* quartets, double* out, size_t out_len,
                              unsigned flags, void* cuda_stream);

/* Boys function F_m(T), m = 0..mmax (mmax <= 4*MAKO_LMAX), for n values T[n] (DEVICE pointers),
 * out[n*(mmax+1)] (DEVICE).  Exposes the device Boys evaluator of the hot path for parity tests. */
mako_status mako_boys(int n, const double* T, int mmax, double* out, void* cuda_stream);

/* thread-local message for the last non-OK status returned on this thread */
const char* mako_last_error(void);
/* library version string */
const char* mako_version(void);

#ifdef __cplusplus
}
#endif
#endif /* MAKO_H */
