// mako_state.h -- host-side state behind the opaque handles of include/mako.h.
#pragma once

#include <map>
#include <memory>
#include <string>
#include <vector>

#include "mako_internal.h"

namespace mako {

// thread-local error message
void set_error(const std::string& msg);
mako_status fail(mako_status st, const std::string& msg);
const char* last_error_cstr();

// owning device buffer (cudaMalloc / cudaFree)
struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
  DevBuf() = default;
  DevBuf(const DevBuf&) = delete;
  DevBuf& operator=(const DevBuf&) = delete;
  DevBuf(DevBuf&& o) noexcept : p(o.p), bytes(o.bytes) { o.p = nullptr; o.bytes = 0; }
  DevBuf& operator=(DevBuf&& o) noexcept {
    if (this != &o) {
      release();
      p = o.p; bytes = o.bytes;
      o.p = nullptr; o.bytes = 0;
    }
    return *this;
  }
  ~DevBuf();
  mako_status alloc(size_t nbytes);
  template <class T> T* as() const { return static_cast<T*>(p); }
  void release();
};

// one bucket (la >= lb) of shell pairs with device-resident primitive-pair data
struct PairBucket {
  int la = 0, lb = 0;
  std::vector<int> shA, shB;       // host copies
  std::vector<double> Q;           // host copy (sorted descending in a screened set)
  std::vector<int> poff;           // [n+1]
  std::vector<int> seg;            // [NKGROUP+1] K-group segment starts (screened sets only)
  DevBuf d_shA, d_shB, d_Q, d_poff, d_pdat, d_Ebra, d_Eket;
  DevBuf d_EbraD, d_EketD;         // FP64 m8n8k4 fragment-order copies (DMMA operand loads)
  DevBuf d_EbraF, d_EketF;         // TF32 fragment-order copies (reduced-precision tier, built on demand)
  int n() const { return (int)shA.size(); }
  PairView view() const;
};

struct PairSet {
  PairBucket b[NBUCKET];
};

// per-class plan for one threshold
struct ClassPlan {
  int X = 0, Y = 0;                // bra / ket buckets (X >= Y)
  int KT = 16;                     // kets per task
  bool swap = false;               // transposed execution: task pairs from bucket Y, lanes from X
  int TB = 0, LB = 0;              // task bucket, lane bucket
  long long ntask = 0;             // tasks of the whole class (all shards)
  long long nquartet = 0;
  // non-empty (bra pair, ket K-group) entries, in (bra Q desc, group) order
  std::vector<int> ent_P, kbeg, kend;  // [nent] bra pair, first / one-past-last surviving ket
  std::vector<long long> task_off;     // [nent + 1] task prefix
  std::vector<int> usamp;              // [ntask / TASK_SAMPLE + 1] entry holding task k * TASK_SAMPLE
  std::vector<long long> unit_off;     // [nunit + 1] first task of each bra unit (all entries of one bra pair)
  std::vector<int> unit_P;             // [nunit] bra pair of the unit
  DevBuf d_ent_P, d_kbeg, d_kend, d_task_off, d_usamp, d_unit_off, d_unit_P;
};

struct Plan {
  double thresh = -1.0;
  int nshards = 1;                 // task lengths are sized for the per-shard quartet count
  double tier = 0.0;               // > thresh: reduced-precision tier boundary (0 = FP64 only)
  int KT = 16;
  std::vector<ClassPlan> cls;      // 55 classes (FP64 tier)
  std::vector<ClassPlan> cls_lo;   // 55 classes, TF32 tier (empty plans where the class has no TF32 kernel)
};

}  // namespace mako

struct mako_basis_s {
  int device = 0;
  int natm = 0;
  std::vector<int> Z;
  std::vector<double> axyz;
  int nshell = 0, nbf = 0, pure = 1;
  std::vector<int> atom, l, nprim, poff, ao;
  std::vector<double> sxyz;     // [nshell*3] shell centres
  std::vector<double> exps, cn; // exponents; coefficient x primitive norm x contraction renorm
  mako::DevBuf d_ao, d_sxyz, d_l, d_poff, d_exps, d_cn, d_sph, d_boys;
  std::vector<int> sph_off;     // offset of each l's [2l+1][ncart] table in d_sph
};

struct mako_pairs_s {
  mako_basis basis = nullptr;   // not owned; must outlive the pairs
  double tau = 0.0;
  mako::PairSet set;
  mako::Plan plan;                       // current plan
  std::vector<mako::Plan> plan_cache;    // recently used plans of other thresholds (density screening)
  mako::DevBuf d_counters;      // [2 * NCLASS] task counters (FP64 tier, TF32 tier)
  mako::DevBuf d_dsh;           // [nshell * nshell] float: max |D| per shell block (density screening)
  mako::DevBuf d_dmax;          // [1] double: max |D| (density screening)
  mako::DevBuf d_jk_scratch;    // [2 * nbf * nbf] accumulators of MAKO_JK_ACCUMULATE builds
  int nsm = 0;                  // SM count of the pairs' device (task-length sizing)
  // profiling (mako_profile_enable / read)
  bool prof = false;
  // concurrent class launches: internal streams forked from / joined to the caller's stream
  std::vector<void*> streams;       // cudaStream_t
  void* ev_fork = nullptr;          // cudaEvent_t
  std::vector<void*> ev_join;       // cudaEvent_t per internal stream
  std::vector<std::pair<int, std::pair<void*, void*>>> prof_events;  // (class, (start, stop)) cudaEvent_t
  ~mako_pairs_s();
};

namespace mako {
// host helpers implemented in basis.cpp
void spherical_tables(std::vector<double>& tab, std::vector<int>& off);   // recurrence-derived
void boys_table(std::vector<double>& tab);                                // composite Gauss-Legendre
// pair-set construction (pairs.cu)
mako_status build_pair_set(const mako_basis_s* B, const std::vector<int> (&A)[NBUCKET],
                           const std::vector<int> (&Bsh)[NBUCKET], PairSet& out, void* stream);
mako_status compute_schwarz(const mako_basis_s* B, PairSet& set, void* stream);
mako_status ensure_lowp(PairSet& set, void* stream);   // TF32 operand copies of every bucket
// class launches (eri_kernels*.cu)
mako_status launch_jk_class(int X, int Y, const JKArgs& a, void* stream, int* nlaunch);
mako_status launch_batch_class(int X, int Y, const BatchArgs& a, void* stream);
bool class_has_lowp(int X, int Y);
// class index (X >= Y) in 0..54
inline int class_index(int X, int Y) { return X * (X + 1) / 2 + Y; }
inline int bucket_la(int b) { int la = 0; while ((la + 1) * (la + 2) / 2 <= b) ++la; return la; }
inline int bucket_lb(int b) { int la = bucket_la(b); return b - la * (la + 1) / 2; }
}  // namespace mako
