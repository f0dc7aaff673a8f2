// cusfft.cu — plan construction, launch sequence and the C ABI declared in
// include/cusfft.h.  Host code runs only at plan time and to enqueue work;
// every step of the transform runs in the kernels of exec_kernels.cuh,
// fft.cuh and tail.cuh.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>  // types only: the library is opened with dlopen when a plan asks for it

#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <string>
#include <utility>
#include <vector>

#include "../../include/cusfft.h"
#include "plan_kernels.cuh"
#include "exchange.cuh"

using namespace cusfft;

namespace {

constexpr uint32_t kMagic = 0x5FF7B200u;
thread_local int g_last_cuda_error = 0;
thread_local int g_last_nccl_error = 0;

#define CK(expr)                                  \
  do {                                            \
    cudaError_t e_ = (expr);                      \
    if (e_ != cudaSuccess) {                      \
      g_last_cuda_error = (int)e_;                \
      return e_ == cudaErrorMemoryAllocation ? CUSFFT_ALLOC : CUSFFT_CUDA; \
    }                                             \
  } while (0)

#define CKL()                                     \
  do {                                            \
    cudaError_t e_ = cudaGetLastError();          \
    if (e_ != cudaSuccess) {                      \
      g_last_cuda_error = (int)e_;                \
      return CUSFFT_CUDA;                         \
    }                                             \
  } while (0)

#define TRY(expr)              \
  do {                         \
    int rc_ = (expr);          \
    if (rc_ != CUSFFT_SUCCESS) \
      return rc_;              \
  } while (0)

bool is_pow2(int64_t v) { return v > 0 && (v & (v - 1)) == 0; }
int ilog2(int64_t v) {
  int l = 0;
  while ((int64_t(1) << l) < v) ++l;
  return l;
}

// SplitMix64 (Steele, Lea, Flood 2014): the seeded generator of the draws
// (DESIGN.md §3 [Z-PRNG]).  The paper only says "a <- random() mod n" (L146).
struct SplitMix64 {
  uint64_t s;
  uint64_t next() {
    s += 0x9E3779B97F4A7C15ull;
    uint64_t z = s;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
  }
};

int64_t gcd64(int64_t a, int64_t b) {
  while (b) {
    int64_t t = a % b;
    a = b;
    b = t;
  }
  return a;
}

// a^-1 mod n by the extended Euclidean algorithm (Alg. 1 line 8, L153).
int64_t inverse_mod(int64_t a, int64_t n) {
  int64_t r0 = n, r1 = a % n, t0 = 0, t1 = 1;
  while (r1) {
    int64_t q = r0 / r1, tmp;
    tmp = r0 - q * r1; r0 = r1; r1 = tmp;
    tmp = t0 - q * t1; t0 = t1; t1 = tmp;
  }
  return ((t0 % n) + n) % n;
}

double binom_tail(int L, double p, int T) {  // P[Binomial(L, p) >= T]
  double s = 0.0;
  for (int v = T; v <= L; ++v) {
    double c = 1.0;
    for (int i = 0; i < v; ++i) c = c * (L - i) / (i + 1);
    s += c * std::pow(p, v) * std::pow(1.0 - p, L - v);
  }
  return s;
}

// ---- NCCL, opened at run time (plans made with an ncclUniqueId only) ----
struct NcclApi {
  bool tried = false, ok = false;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
};
std::mutex g_nccl_mu;
NcclApi g_nccl;

const NcclApi* nccl_api() {
  std::lock_guard<std::mutex> lk(g_nccl_mu);
  if (!g_nccl.tried) {
    g_nccl.tried = true;
    // the process's NCCL if one is loaded already (e.g. PyTorch's), else the system one
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (h) {
      g_nccl.CommInitRank = (decltype(g_nccl.CommInitRank))dlsym(h, "ncclCommInitRank");
      g_nccl.CommDestroy = (decltype(g_nccl.CommDestroy))dlsym(h, "ncclCommDestroy");
      g_nccl.GetUniqueId = (decltype(g_nccl.GetUniqueId))dlsym(h, "ncclGetUniqueId");
      g_nccl.AllGather = (decltype(g_nccl.AllGather))dlsym(h, "ncclAllGather");
      g_nccl.AllReduce = (decltype(g_nccl.AllReduce))dlsym(h, "ncclAllReduce");
      g_nccl.ok = g_nccl.CommInitRank && g_nccl.CommDestroy && g_nccl.GetUniqueId && g_nccl.AllGather &&
                  g_nccl.AllReduce;
    }
  }
  return g_nccl.ok ? &g_nccl : nullptr;
}

}  // namespace

// A filter of the plan (DESIGN.md §3 [Z1]): group 0 filters the location loops
// r < L_loc, group 1 the estimation-only loops; one group when the
// two parameter sets are equal (or the caller supplies taps).
struct Filter {
  double tolerance = 0, lobefrac = 0;
  int w = 0, R = 0;                 // taps, rounds R = ceil(w / B)
  double* d_taps = nullptr;         // [R B] zero-padded past w
  double* d_taps_perm = nullptr;    // [R B] tile-permuted (fused fold + FFT pass 1 layout)
  double2* d_ghat = nullptr;        // [nb + 1] G^(q), q = -nb/2 .. nb/2
  double2* d_ginv = nullptr;        // [nb + 1] 1 / G^(q)
};

struct cusfft_plan_s {
  uint32_t magic = kMagic;
  int64_t n = 0, k = 0, B = 0, nb = 0;
  int L = 0, Lg = 0, rank = 0, world = 1;
  // Loop layout: loop sharding uses (lrank, lworld) = (rank, world); a
  // signal-sharded plan runs every loop, (lrank, lworld) = (0, 1),
  // on its slice x[xlo, xlo + xspan) and sums partial spectra in the exchange.
  bool xshard = false;
  int lrank = 0, lworld = 1;
  uint32_t xlo = 0, xspan = 0;
  cusfft_params prm{};            // prm.taps points at user_taps (plan-owned copy) or is NULL
  std::vector<double> user_taps;  // host copy of caller-supplied taps (clones are built from it)
  int log2nb = 0, num = 0, Lloc = 0, T = 0, max_hits = 0;
  int Jcap = 0;  // winner-list capacity per loop (num, or B in THRESHOLD mode)
  int B1 = 1, B2 = 1, logB1 = 0, logB2 = 0;
  int kp2 = 1;
  int nfilt = 1;
  Filter filt[2];
  int wmax = 0;
  std::vector<SlotParam> slots_h;            // slot order
  std::vector<int64_t> a_r, sigma_r, tau_r;  // loop order
  std::vector<int> loc_slots_h, sel_slots_h;
  int nloc_local = 0;                        // local slots [0, nloc_local) are location loops
  RecLayout lay{};
  bool fused1 = false;                       // fold fused with FFT pass 1 (B1 in [64, 256])
  // staged gather: address-sorted gather schedule of this rank
  bool staged = false;
  int stage_ibits = 0;
  int64_t stage_total = 0;                   // gathers of this rank (sum of the local slots' w)
  uint32_t* d_code = nullptr;                // [stage_total] (local slot << ibits | i) in address order
  uint32_t* d_row0 = nullptr;                // [Lg] first staging row of each local slot
  std::vector<uint32_t> row0_h;              // same, host (+ total rows at [Lg]); relative to the slot's group
  // Stage groups (plans whose staging of all slots would not fit L2, e.g. C4): consecutive local
  // slots [grp_s[g], grp_s[g + 1]) whose gathers are sorted, staged and folded together, one
  // group after the other through one staging buffer; one group = the whole-plan staging.
  std::vector<int> grp_s;
  std::vector<int64_t> grp_off;              // first schedule word of each group (+ total at the end)
  bool grp_abs = false;                      // groups keep their own staging rows (all of it fits L2)
  double2* d_staging = nullptr;              // [rows][B]
  int stage_grid = 1;
  // gather 2 (ablation): the paper's remap + execute kernels on concurrent streams
  bool remap = false;
  double2* d_remap = nullptr;                // [nrm][B] one reordered chunk A' per stream
  std::vector<cudaStream_t> rm_st;
  std::vector<cudaEvent_t> rm_ev;            // [0] fork, [1 + i] join of stream i
  bool p2_ms = true;                         // phase 2 in the multi-slot form (k_fold_fft1_ms, R <= 16)
  int p2_spc = 2;                            // phase-2 slots per CTA (taps reused across them; 1 / 4 slower)
  int fork_at = 1;                           // estimation branch forks after phase 1 (0) or after the location phase 2 (1, measured ~0.5 us faster)
  bool setaside = false;                     // holds a reference on the device's persisting-L2 set-aside
  int64_t sectors = 0;                       // distinct 32-B sectors of x gathered by this rank
  double2* d_tw = nullptr;
  double2* d_ph_hi = nullptr;     // e^{-2 pi i (j << plo) / n}: the estimation's phase, high bits
  double2* d_ph_lo = nullptr;     // e^{-2 pi i j / n}, j < 2^plo: low bits
  int plo = 0;
  SlotParam* d_slots = nullptr;
  uint32_t* d_loc_sigma = nullptr;
  double2* d_u = nullptr;
  double2* d_v = nullptr;
  uint8_t* d_records = nullptr;
  uint64_t* d_keys = nullptr;     // [n_sel][B] cutoff keys of this rank's location loops
  uint32_t* d_hist = nullptr;     // [n_sel][4096] top-digit histograms (zero block)
  int* d_key_index = nullptr;     // [Lg] local slot -> selection index or -1
  uint32_t* d_ohist = nullptr;    // [4096] top-digit histogram of the output keys (zero block)
  bool fft2sel = true;             // location slots' FFT pass 2 fused with the cutoff when the shape allows (use_fft2_select)
  bool sel_cluster = false;       // k_select_cluster (256 <= B <= 65536, EXACT / THRESHOLD modes)
  int select1_smem = 0;
  // fused vote + estimate + output (k_tail) when its table fits shared memory
  // shard_mode 2 (two all-gathers, exchange.cuh): candidate records, then per-loop estimates
  bool mode2 = false;
  int cmax = 0;                   // candidate records per rank slice (location loops of the busiest rank)
  int64_t crec_bytes = 0;         // one candidate record: bitmap | count | J (the record's tail)
  uint8_t* d_cand = nullptr;      // [world][cmax][crec_bytes]
  double2* d_x2 = nullptr;        // [world][max_hits][Lg] per-loop estimates
  int* d_hits2 = nullptr;          // [max_hits] the hit list in ascending order (k_rank_est)
  int tail_esz = 0;               // bytes per vote-table element (1 / 2 / 4), 0: the k_vote / k_estimate / k_output chain
  int tail_smem = 0, tail_qoff = 0, tail_grid = 1;
  bool pk_direct = false;         // the cluster cutoff ORs its winners into k_tail's table (d_pk, zero block)
  uint32_t* d_pk = nullptr;
  uint32_t* d_pkb = nullptr;      // otherwise (fused tail): the table built once by k_pk_build before k_tail
  int vote_smem = 0, vote_grid = 1, est_grid = 1, output_smem = 0;
  int* d_hits = nullptr;
  double2* d_hit_vals = nullptr;
  uint64_t* d_hit_keys = nullptr;
  double2* d_per_loop = nullptr;
  int* d_zero = nullptr;   // per-execution block, zeroed by the first kernel of each execution:
  int nzero = 0;           //   flags[8] | hist0[n_sel][4096] | ohist[4096] | pad [4] | pk
  int* d_flags = nullptr;  // [0] hit_count (unsigned), [1] overflow, [2] select mismatch, [3] output mismatch
  double2* d_xbuf = nullptr;
  int64_t* d_locs_buf = nullptr;
  double2* d_vals_buf = nullptr;
  cudaStream_t stream = nullptr;
  bool own_stream = false;        // clone plans (batched execution) own their stream
  int device = 0;
  int sms = 148;
  int timing = 0;          // 1: direct launches with events between the stages; 2: events inside the graph
  cudaEvent_t ev[8] = {};  // stage boundaries 0..6; [7] after phase 1 of the staged fold
  bool ev_made = false;
  ncclComm_t comm = nullptr;      // library-owned exchange (cusfft_plan_dist with an ncclUniqueId)
  bool use_graph = true;
  cudaStream_t cap_stream = nullptr, cap_stream2 = nullptr;
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  int stage_limit = 6;
  int cur_prio = 0, prio_hi = 0, prio_lo = 0;  // launch priorities (two-branch graph)
  struct GraphEntry {
    int lim = -1, tmode = 0;
    const void* a = nullptr;
    const void* b = nullptr;
    const void* c = nullptr;
    cudaGraphExec_t exec = nullptr;
  } g_local, g_mid, g_finish;
  // whole-transform graphs by (x, locs, vals): up to kGraphCache, least recently used replaced
  std::vector<GraphEntry> g_cache;
  std::vector<uint64_t> g_used;
  uint64_t g_tick = 0;
  // batched execution (cusfft_execute_batch): depth-1 clones of this plan, each on its own stream
  std::vector<cusfft_plan_s*> subs;
  std::vector<cudaEvent_t> sub_ev;  // [depth] join events (+ fork event at the end)

  int filt_of_slot(int s) const { return (nfilt > 1 && (int)slots_h[s].loop >= Lloc) ? 1 : 0; }
  int filt_of_local(int i) const { return filt_of_slot(lrank * Lg + i); }
};

constexpr size_t kGraphCache = 64;

namespace {

bool valid_plan(cusfft_plan_t p) { return p && p->magic == kMagic; }

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

// Device-wide persisting-L2 set-aside (cudaLimitPersistingL2CacheSize), shared
// by the plans of a device that ask for it (params.l2_persist = 1): raised to
// the largest request while any such plan lives, restored to the value found
// before the first when the last one is destroyed (include/cusfft.h).
struct SetAside {
  int refs = 0;
  size_t orig = 0, cur = 0;
};
std::mutex g_setaside_mu;
SetAside g_setaside[64];

void setaside_acquire(int dev, size_t bytes) {
  std::lock_guard<std::mutex> lk(g_setaside_mu);
  SetAside& a = g_setaside[dev & 63];
  if (a.refs++ == 0) {
    cudaDeviceGetLimit(&a.orig, cudaLimitPersistingL2CacheSize);
    a.cur = a.orig;
  }
  if (bytes > a.cur && cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, bytes) == cudaSuccess) a.cur = bytes;
  cudaGetLastError();
}

void setaside_release(int dev) {
  std::lock_guard<std::mutex> lk(g_setaside_mu);
  SetAside& a = g_setaside[dev & 63];
  if (a.refs > 0 && --a.refs == 0 && a.cur != a.orig) {
    cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, a.orig);
    cudaGetLastError();
    a.cur = a.orig;
  }
}

void free_plan(cusfft_plan_t p) {
  for (auto& f : p->filt) {
    if (f.d_taps) cudaFree(f.d_taps);
    if (f.d_taps_perm) cudaFree(f.d_taps_perm);
    if (f.d_ghat) cudaFree(f.d_ghat);
    if (f.d_ginv) cudaFree(f.d_ginv);
  }
  void* ptrs[] = {p->d_code, p->d_row0, p->d_staging, p->d_tw, p->d_ph_hi, p->d_ph_lo, p->d_slots, p->d_loc_sigma, p->d_u, p->d_v,
                  p->d_records, p->d_keys, p->d_zero, p->d_key_index, p->d_hits, p->d_hit_vals, p->d_hit_keys,
                  p->d_per_loop, p->d_xbuf, p->d_locs_buf, p->d_vals_buf, p->d_cand, p->d_x2, p->d_hits2, p->d_pkb};
  for (void* q : ptrs)
    if (q) cudaFree(q);
  if (p->ev_made)
    for (auto& e : p->ev) cudaEventDestroy(e);
  for (auto* g : {&p->g_local, &p->g_mid, &p->g_finish})
    if (g->exec) cudaGraphExecDestroy(g->exec);
  for (auto& g : p->g_cache)
    if (g.exec) cudaGraphExecDestroy(g.exec);
  for (auto* sp : p->subs) free_plan(sp);
  for (auto e : p->sub_ev) cudaEventDestroy(e);
  if (p->comm) {
    if (const NcclApi* api = nccl_api()) api->CommDestroy(p->comm);
  }
  if (p->own_stream && p->stream) cudaStreamDestroy(p->stream);
  if (p->cap_stream) cudaStreamDestroy(p->cap_stream);
  if (p->cap_stream2) cudaStreamDestroy(p->cap_stream2);
  if (p->ev_fork) cudaEventDestroy(p->ev_fork);
  if (p->ev_join) cudaEventDestroy(p->ev_join);
  for (auto st : p->rm_st) cudaStreamDestroy(st);
  for (auto e : p->rm_ev) cudaEventDestroy(e);
  if (p->d_remap) cudaFree(p->d_remap);
  if (p->setaside) setaside_release(p->device);
  p->magic = 0;
  delete p;
}

int validate(int64_t n, int64_t k, int64_t B, int32_t L, const cusfft_params& q, int rank, int world) {
  if (!is_pow2(n) || n < 16 || n > (int64_t(1) << 31)) return CUSFFT_INVALID_N;
  if (!is_pow2(B) || B < 2 || B >= n) return CUSFFT_INVALID_B;
  if (L < 1 || L > kMaxLoops) return CUSFFT_INVALID_LOOPS;
  if (q.loc_loops > kMaxLoc) return CUSFFT_INVALID_LOOPS;
  if (world < 1 || rank < 0 || rank >= world) return CUSFFT_INVALID_LOOPS;
  if (q.shard_mode < 0 || q.shard_mode > 2) return CUSFFT_INVALID_PARAM;
  // shard_mode 2: the hits are ranked by counting (quadratic in them), the median holds 2 values per lane
  if (q.shard_mode == 2 && (q.max_hits > 32768 || L > kMedMaxL)) return CUSFFT_INVALID_PARAM;
  if (q.shard_mode == 1 && world > 1) {
    if (n % world) return CUSFFT_INVALID_PARAM;
  } else if (L % world) {
    return CUSFFT_INVALID_LOOPS;
  }
  if (q.loc_loops < 1 || q.loc_loops > L || q.vote_threshold < 1 || q.vote_threshold > q.loc_loops)
    return CUSFFT_INVALID_LOOPS;
  if (k < 1 || k > 8192 || q.num_select < k || q.num_select > B) return CUSFFT_INVALID_K;
  if (q.taps) {
    if (q.num_taps < 1 || q.num_taps > (int64_t(1) << 30)) return CUSFFT_INVALID_PARAM;
  } else {
    if (q.filter != CUSFFT_FILTER_DOLPH_CHEBYSHEV && q.filter != CUSFFT_FILTER_GAUSSIAN) return CUSFFT_INVALID_PARAM;
    if (!(q.tolerance > 0.0 && q.tolerance < 1.0)) return CUSFFT_INVALID_PARAM;
    if (!(q.lobefrac > 0.0 && q.lobefrac < 0.5)) return CUSFFT_INVALID_PARAM;
    if (!(q.loc_tolerance == 0.0 || (q.loc_tolerance > 0.0 && q.loc_tolerance < 1.0))) return CUSFFT_INVALID_PARAM;
    if (!(q.loc_lobefrac == 0.0 || (q.loc_lobefrac > 0.0 && q.loc_lobefrac < 0.5))) return CUSFFT_INVALID_PARAM;
    if (q.box_width < 1 || q.box_width > n || (q.box_width % 2) == 0) return CUSFFT_INVALID_PARAM;
  }
  if (q.max_hits < 1 || q.max_hits > (int64_t(1) << 30)) return CUSFFT_INVALID_PARAM;
  if (q.cutoff_mode < CUSFFT_CUTOFF_EXACT || q.cutoff_mode > CUSFFT_CUTOFF_THRESHOLD) return CUSFFT_INVALID_PARAM;
  if (q.cutoff_mode == CUSFFT_CUTOFF_SORT && B > 16384) return CUSFFT_INVALID_PARAM;
  if (q.cutoff_mode == CUSFFT_CUTOFF_THRESHOLD && !(q.cutoff_threshold > 0.0)) return CUSFFT_INVALID_PARAM;
  if (q.tau_mode != 0 && q.tau_mode != 1) return CUSFFT_INVALID_PARAM;
  if (q.l2_persist != 0 && q.l2_persist != 1) return CUSFFT_INVALID_PARAM;
  if (q.gather < 0 || q.gather > 2) return CUSFFT_INVALID_PARAM;
  if (q.gather == 2 && q.shard_mode == 1) return CUSFFT_INVALID_PARAM;  // the remap ablation folds whole signals
  return CUSFFT_SUCCESS;
}

// w = floor(acosh(1/delta) / (pi lambda)) (Dolph-Chebyshev) or
// floor(2 ln(1/delta) / (pi lambda)) (Gaussian), forced odd [Z1].
int64_t filter_len(int filter, double tol, double lob) {
  const double pi = 3.14159265358979323846;
  int64_t w;
  if (filter == CUSFFT_FILTER_DOLPH_CHEBYSHEV)
    w = (int64_t)std::floor(std::acosh(1.0 / tol) / (pi * lob));
  else
    w = (int64_t)std::floor(2.0 * std::log(1.0 / tol) / (pi * lob));
  if (w % 2 == 0) --w;
  return w;
}

template <class T>
int dalloc(T** ptr, size_t count) {
  if (count == 0) count = 1;
  CK(cudaMalloc((void**)ptr, count * sizeof(T)));
  return CUSFFT_SUCCESS;
}

int upload(void* dst, const void* src, size_t bytes) {
  CK(cudaMemcpy(dst, src, bytes, cudaMemcpyHostToDevice));
  return CUSFFT_SUCCESS;
}

// Taps g_i (window x box, normalised to sum 1), G^ and, for fused plans, the
// tile-permuted tap layout of one filter (plan_kernels.cuh; DESIGN.md §3 [Z1]).
int build_filter(cusfft_plan_t P, Filter& F) {
  const cusfft_params& q = P->prm;
  const int w = F.w;
  const int64_t B = P->B;
  const int padded = F.R * (int)B;
  const int c = (w - 1) / 2;
  cudaStream_t st = P->stream;
  TRY(dalloc(&F.d_taps, (size_t)padded));
  TRY(dalloc(&F.d_ghat, (size_t)P->nb + 1));
  TRY(dalloc(&F.d_ginv, (size_t)P->nb + 1));
  if (q.taps) {
    CK(cudaMemsetAsync(F.d_taps, 0, (size_t)padded * sizeof(double), st));
    CK(cudaMemcpyAsync(F.d_taps, q.taps, (size_t)w * sizeof(double), cudaMemcpyHostToDevice, st));
  } else {
    double* win = nullptr;
    double* pj = nullptr;
    TRY(dalloc(&win, (size_t)c + 1));
    if (q.filter == CUSFFT_FILTER_DOLPH_CHEBYSHEV) {
      TRY(dalloc(&pj, (size_t)c + 1));
      const double x0 = std::cosh(std::acosh(1.0 / F.tolerance) / (double)(w - 1));
      k_cheb_samples<<<(c + 256) / 256, 256, 0, st>>>(pj, w, x0);
      CKL();
      k_dc_window<<<c + 1, 256, 0, st>>>(pj, win, w);
      CKL();
    } else {
      const double s = (double)c / std::sqrt(2.0 * std::log(1.0 / F.tolerance));
      k_gauss_window<<<(c + 256) / 256, 256, 0, st>>>(win, w, s);
      CKL();
    }
    k_taps<<<(padded + 255) / 256, 256, 0, st>>>(win, F.d_taps, w, padded, P->n, q.box_width);
    CKL();
    k_normalize<<<1, 1024, 0, st>>>(F.d_taps, w);
    CKL();
    CK(cudaStreamSynchronize(st));
    cudaFree(win);
    if (pj) cudaFree(pj);
  }
  k_ghat<<<(int)P->nb + 1, 256, 0, st>>>(F.d_taps, F.d_ghat, w, P->n, (int)P->nb);
  CKL();
  k_ginv<<<(int)((P->nb + 256) / 256), 256, 0, st>>>(F.d_ghat, F.d_ginv, (int)P->nb + 1);
  CKL();
  if (P->fused1) {  // taps_perm[rr B + cta 256 + t] = g[j(cta, t) + rr B], j = c + B2 j1
    std::vector<double> g((size_t)padded), gp((size_t)padded);
    CK(cudaMemcpy(g.data(), F.d_taps, (size_t)padded * sizeof(double), cudaMemcpyDeviceToHost));
    const int C = 256 / P->B1;
    for (int64_t rr = 0; rr < F.R; ++rr)
      for (int64_t cta = 0; cta < B / 256; ++cta)
        for (int t = 0; t < 256; ++t) {
          const int64_t cc = cta * C + t / P->B1, j1 = t % P->B1;
          gp[(size_t)(rr * B + cta * 256 + t)] = g[(size_t)(rr * B + cc + (int64_t)P->B2 * j1)];
        }
    TRY(dalloc(&F.d_taps_perm, (size_t)padded));
    TRY(upload(F.d_taps_perm, gp.data(), (size_t)padded * sizeof(double)));
  }
  return CUSFFT_SUCCESS;
}

// Kernel launch carrying an explicit scheduling priority (stream priorities
// are not captured into graph kernel nodes, the launch attribute is) and,
// with g_pdl, programmatic dependent launch (every hot kernel begins with
// pdl_wait(), so it may be launched while its predecessor drains).
thread_local bool g_pdl = false;

template <typename... KArgs, typename... Args>
cudaError_t launch_k(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, int prio,
                     Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = prio;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = g_pdl ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// Batched M-point FFT passes: 512 elements per CTA for M < 512 except M = 256
// (measured best at C3 against 256 and 1024), one sequence per CTA above.
// (M = 256, C4's row FFTs: 1024 elements per CTA, 17.8 vs 21.5 µs at 512 and 21.4 at 2048;
// profiles/r02_stage_ab.md)
template <int M>
constexpr int fft_E() { return M == 256 ? 1024 : M < 512 ? 512 : M; }

template <int M>
cudaError_t launch_fft_t(const FftPassArgs& a, cudaStream_t st, int prio) {
  constexpr int E = fft_E<M>();
  constexpr int NSEQ = E / M;
  const int grid = (a.total_seq + NSEQ - 1) / NSEQ;
  return launch_k(k_fft<M, E, 128>, dim3(grid), dim3(128), fft_smem_bytes(E), st, prio, a);
}

cudaError_t launch_fft(int M, const FftPassArgs& a, cudaStream_t st, int prio = 0) {
  switch (M) {
    case 2: return launch_fft_t<2>(a, st, prio);
    case 4: return launch_fft_t<4>(a, st, prio);
    case 8: return launch_fft_t<8>(a, st, prio);
    case 16: return launch_fft_t<16>(a, st, prio);
    case 32: return launch_fft_t<32>(a, st, prio);
    case 64: return launch_fft_t<64>(a, st, prio);
    case 128: return launch_fft_t<128>(a, st, prio);
    case 256: return launch_fft_t<256>(a, st, prio);
    case 512: return launch_fft_t<512>(a, st, prio);
    case 1024: return launch_fft_t<1024>(a, st, prio);
    case 2048: return launch_fft_t<2048>(a, st, prio);
    case 4096: return launch_fft_t<4096>(a, st, prio);
    default: return cudaErrorInvalidValue;
  }
}

template <int M>
cudaError_t set_fft_attr() {
  return cudaFuncSetAttribute(k_fft<M, fft_E<M>(), 128>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              fft_smem_bytes(fft_E<M>()));
}

cudaError_t set_fft_attrs() {
  cudaError_t e = cudaSuccess;
  cudaError_t r[] = {set_fft_attr<2>(), set_fft_attr<4>(), set_fft_attr<8>(), set_fft_attr<16>(),
                     set_fft_attr<32>(), set_fft_attr<64>(), set_fft_attr<128>(), set_fft_attr<256>(),
                     set_fft_attr<512>(), set_fft_attr<1024>(), set_fft_attr<2048>(), set_fft_attr<4096>()};
  for (cudaError_t x : r)
    if (x != cudaSuccess) e = x;
  return e;
}

// Allow `want` bytes of dynamic shared memory, capped at what the device leaves
// next to the kernel's static shared memory.
template <typename K>
cudaError_t set_dyn_smem(K* kern, int want, int optin) {
  cudaFuncAttributes fa{};
  cudaError_t e = cudaFuncGetAttributes(&fa, kern);
  if (e != cudaSuccess) return e;
  const int cap = optin - (int)fa.sharedSizeBytes;
  return cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, std::min(want, cap));
}

// k_tail instantiation of a plan: vote-table element (tail_esz), estimation
// lanes per hit (L <= 16: 16), compile-time L_loc = 8 for the default plans.
using TailKernel = void (*)(TailArgs);
TailKernel tail_kernel(int esz, int L, int Lloc) {
  const bool seg = L <= 16;
  if (esz == 1 && Lloc == 8) return seg ? k_tail<uint8_t, 16, 8> : k_tail<uint8_t, 32, 8>;
  if (esz == 1) return seg ? k_tail<uint8_t, 16, 0> : k_tail<uint8_t, 32, 0>;
  if (esz == 2) return seg ? k_tail<uint16_t, 16, 0> : k_tail<uint16_t, 32, 0>;
  return seg ? k_tail<uint32_t, 16, 0> : k_tail<uint32_t, 32, 0>;
}
// The vote-only instantiation (shard_mode 2: each rank estimates its own loops afterwards).
TailKernel tail_vote_kernel(int esz, int Lloc) {
  if (esz == 1 && Lloc == 8) return k_tail<uint8_t, 16, 8, false>;
  if (esz == 1) return k_tail<uint8_t, 16, 0, false>;
  if (esz == 2) return k_tail<uint16_t, 16, 0, false>;
  return k_tail<uint32_t, 16, 0, false>;
}

int make_plan(cusfft_plan_t* out, int64_t n, int64_t k, int64_t B, int32_t L, const cusfft_params* pin, int rank,
              int world, const void* nccl_id) {
  if (!out) return CUSFFT_NULL_PTR;
  cusfft_params q;
  if (pin) {
    q = *pin;
  } else {
    int rc = cusfft_params_default(&q, n, k, B);
    if (rc) return rc;
  }
  if (!pin || q.loc_loops == 0) q.loc_loops = std::min<int32_t>(L, 8);
  if (!pin || q.vote_threshold == 0) q.vote_threshold = q.loc_loops / 2 + 1;
  if (q.num_select == 0) q.num_select = (int32_t)k;
  if (q.max_hits == 0) {
    const double pr = (double)q.num_select / (double)B;
    double e = (double)n * binom_tail(q.loc_loops, pr, q.vote_threshold) + (double)k;
    int64_t mh = std::max<int64_t>(16384, (int64_t)(4.0 * e));
    q.max_hits = std::min<int64_t>(mh, std::min<int64_t>(n, int64_t(1) << 30));
  }
  TRY(validate(n, k, B, L, q, rank, world));
  int ndev = 0;
  CK(cudaGetDeviceCount(&ndev));
  if (ndev < 1) {
    g_last_cuda_error = (int)cudaErrorNoDevice;
    return CUSFFT_CUDA;
  }
  int dev = q.device;
  if (dev < 0) CK(cudaGetDevice(&dev));
  if (dev >= ndev) return CUSFFT_INVALID_PARAM;
  DeviceGuard guard(dev);
  const NcclApi* api = nullptr;
  if (nccl_id) {
    api = nccl_api();
    if (!api) return CUSFFT_NCCL;
  }

  cusfft_plan_t P = new (std::nothrow) cusfft_plan_s();
  if (!P) return CUSFFT_ALLOC;
  auto fail = [&](int code) {
    free_plan(P);
    return code;
  };
  P->n = n; P->k = k; P->B = B; P->L = L; P->prm = q; P->rank = rank; P->world = world;
  if (q.taps) {  // the caller keeps ownership of its array: keep a copy (cusfft_set_pipeline clones read it)
    P->user_taps.assign(q.taps, q.taps + q.num_taps);
    P->prm.taps = P->user_taps.data();
  }
  P->device = dev;
  cudaDeviceGetAttribute(&P->sms, cudaDevAttrMultiProcessorCount, dev);
  P->nb = n / B;
  P->log2nb = ilog2(P->nb);
  P->xshard = world > 1 && q.shard_mode == 1;
  P->lrank = P->xshard ? 0 : rank;
  P->lworld = P->xshard ? 1 : world;
  P->xspan = (uint32_t)(P->xshard ? n / world : n);
  P->xlo = P->xshard ? (uint32_t)rank * P->xspan : 0u;
  P->Lg = L / P->lworld;
  P->num = q.num_select;
  P->Lloc = q.loc_loops;
  P->T = q.vote_threshold;
  P->max_hits = (int)q.max_hits;
  if (const char* e = std::getenv("CUSFFT_NO_GRAPH")) P->use_graph = !(e[0] == '1');                    // A/B (measurement)
  if (const char* e = std::getenv("CUSFFT_P2_MS")) P->p2_ms = std::atoi(e) != 0;                         // A/B (measurement)
  if (const char* e = std::getenv("CUSFFT_P2_SPC")) P->p2_spc = std::max(1, std::min(8, std::atoi(e)));  // A/B (measurement)
  if (const char* e = std::getenv("CUSFFT_FFT2SEL")) P->fft2sel = std::atoi(e) != 0;                     // A/B (measurement)
  if (const char* e = std::getenv("CUSFFT_FORK")) P->fork_at = std::atoi(e);                                 // A/B (measurement)
  // ---- filters (group 0: location loops; group 1: estimation-only loops)
  {
    const double tl = q.loc_tolerance > 0.0 ? q.loc_tolerance : q.tolerance;
    const double ll = q.loc_lobefrac > 0.0 ? q.loc_lobefrac : q.lobefrac;
    P->filt[0].tolerance = tl;
    P->filt[0].lobefrac = ll;
    P->filt[1].tolerance = q.tolerance;
    P->filt[1].lobefrac = q.lobefrac;
    P->nfilt = (!q.taps && P->Lloc < L && (tl != q.tolerance || ll != q.lobefrac)) ? 2 : 1;
    for (int f = 0; f < P->nfilt; ++f) {
      const int64_t w64 = q.taps ? q.num_taps : filter_len(q.filter, P->filt[f].tolerance, P->filt[f].lobefrac);
      // (a filter longer than the signal would wrap around it: not the paper's flat window, L85)
      if (w64 < 1 || w64 > (int64_t(1) << 30) || w64 > n) return fail(CUSFFT_INVALID_PARAM);
      P->filt[f].w = (int)w64;
      P->filt[f].R = (int)((w64 + B - 1) / B);
      P->wmax = std::max(P->wmax, (int)w64);
    }
  }
  P->stream = nullptr;

  // ---- draws (loop order), Alg. 1, Def. 1
  SplitMix64 rng{q.seed};
  P->a_r.resize(L); P->sigma_r.resize(L); P->tau_r.resize(L);
  for (int r = 0; r < L; ++r) {
    int64_t a = (int64_t)(rng.next() % (uint64_t)n);
    while (gcd64(a, n) != 1) a = (int64_t)(rng.next() % (uint64_t)n);
    P->a_r[r] = a;
    P->sigma_r[r] = inverse_mod(a, n);
    P->tau_r[r] = q.tau_mode ? (int64_t)(rng.next() % (uint64_t)n) : 0;
  }
  // ---- slots: rank g owns loops r = i*lworld + g at slots g*Lg + i
  const int lworld = P->lworld, lrank = P->lrank;
  P->slots_h.resize(L);
  for (int s = 0; s < L; ++s) {
    const int g = s / P->Lg, i = s % P->Lg, r = i * lworld + g;
    P->slots_h[s] = SlotParam{(uint32_t)P->sigma_r[r], (uint32_t)P->tau_r[r], (uint32_t)P->a_r[r], (uint32_t)r};
  }
  for (int i = 0; i < P->Lg; ++i)
    if (i * lworld + lrank < P->Lloc) P->nloc_local = i + 1;  // location loops are a prefix of the local slots
  std::vector<uint32_t> loc_sig;
  for (int s = 0; s < L; ++s) {
    if ((int)P->slots_h[s].loop < P->Lloc) {
      P->loc_slots_h.push_back(s);
      loc_sig.push_back(P->slots_h[s].sigma);
      if (s / P->Lg == lrank) P->sel_slots_h.push_back(s);
    }
  }

  // ---- layout
  auto align256 = [](int64_t v) { return (v + 255) & ~int64_t(255); };
  P->Jcap = q.cutoff_mode == CUSFFT_CUTOFF_THRESHOLD ? (int)B : P->num;
  P->lay.off_bitmap = align256(B * 16);
  P->lay.off_cnt = align256(P->lay.off_bitmap + ((B + 31) / 32) * 4);
  P->lay.off_J = P->lay.off_cnt + 16;
  P->lay.rec_bytes = align256(P->lay.off_J + (int64_t)P->Jcap * 4);
  // one FFT pass (and the direct fold) only below 2048 buckets: B = 2048 = 64 x 32 takes the
  // staged fold with pass 1 inside it (C2: 47.2 -> 37.5 us, C5 k = 50: 49 -> 39 us; its one
  // 2048-point FFT per loop ran on 16 CTAs)
  if (B < 2048) {
    P->B1 = 1; P->B2 = (int)B;
  } else {
    const int lb = ilog2(B);
    P->B1 = 1 << ((lb + 1) / 2);
    P->B2 = (int)(B / P->B1);
  }
  P->logB1 = ilog2(P->B1);
  P->logB2 = ilog2(P->B2);
  P->fused1 = P->B1 > 1 && P->B1 <= 256 && q.gather != 2;  // gather 2: the paper's remap + execute (unfused)
  P->kp2 = 1;
  while (P->kp2 < k) P->kp2 <<= 1;
  int smem_optin = 200 * 1024;
  cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  const int nsel = (int)P->sel_slots_h.size();
  P->sel_cluster = B >= 256 && B <= 65536 && q.cutoff_mode != CUSFFT_CUTOFF_SORT;
  P->select1_smem = 4096 * 4 + 64 * 4 + kSelCap * 12 + (int)((B + 31) / 32) * 4;
  if (!P->sel_cluster && q.cutoff_mode != CUSFFT_CUTOFF_SORT && P->select1_smem > smem_optin)
    return fail(CUSFFT_INVALID_B);
  // ---- fused vote + estimation (k_tail): table element by L_loc, table + queues in smem
  {
    const int esz = P->Lloc <= 8 ? 1 : P->Lloc <= 16 ? 2 : 4;
    const int64_t tab = ((int64_t)B * esz + 15) & ~int64_t(15);
    const int64_t need = tab + (kTailNT / 32) * kTailQ * 2;
    const char* et = std::getenv("CUSFFT_TAIL");  // CUSFFT_TAIL=0: the k_vote / k_estimate chain (tests, A/B)
    // (shard_mode 2 runs it vote-only: each rank estimates its own loops afterwards)
    if (need + 8 * 1024 <= smem_optin && !(et && et[0] == '0')) {  // + k_tail's static smem (hit queue)
      P->tail_esz = esz;
      P->tail_qoff = (int)tab;
      P->tail_smem = (int)need;
    }
  }
  P->vote_smem = P->Lloc * (int)((B + 31) / 32) * 4;
  P->output_smem = output_smem_total(P->kp2);
  if ((!P->tail_esz && P->vote_smem > smem_optin) || P->output_smem + 1024 > smem_optin) return fail(CUSFFT_INVALID_B);
  {
    const int64_t units = (int64_t)(P->Lloc - P->T + 1) * P->num;  // k_vote: one warp per (q0, J) range
    P->vote_grid = (int)std::max<int64_t>(1, std::min<int64_t>((units + 7) / 8, (int64_t)P->sms * 4));
    P->est_grid = std::max(1, std::min((P->max_hits + 7) / 8, P->sms * 4));
  }

  int rc = CUSFFT_SUCCESS;
  if ((rc = dalloc(&P->d_tw, (size_t)B))) return fail(rc);
  if ((rc = dalloc(&P->d_slots, (size_t)L))) return fail(rc);
  if ((rc = dalloc(&P->d_loc_sigma, (size_t)P->Lloc))) return fail(rc);
  if ((rc = dalloc(&P->d_u, (size_t)P->Lg * B))) return fail(rc);
  if (P->B1 > 1 && (rc = dalloc(&P->d_v, (size_t)P->Lg * B))) return fail(rc);
  if ((rc = dalloc(&P->d_records, (size_t)L * P->lay.rec_bytes))) return fail(rc);
  if ((rc = dalloc(&P->d_keys, (size_t)std::max(1, nsel) * B))) return fail(rc);
  {
    // per-execution counters and histograms: one block, zeroed by the first kernel
    P->pk_direct = P->tail_esz && P->sel_cluster && P->sel_slots_h == P->loc_slots_h && B % 32 == 0 &&
                   q.cutoff_mode != CUSFFT_CUTOFF_SORT;
    const int base = 8 + nsel * 4096 + 4096 + 4;
    const int pk_off = (base + 3) & ~3;  // 16-B aligned (uint4 copies)
    P->nzero = P->pk_direct ? pk_off + (int)(((int64_t)B * P->tail_esz + 15) / 16) * 4 : base;
    if ((rc = dalloc(&P->d_zero, (size_t)P->nzero))) return fail(rc);
    P->d_flags = P->d_zero;
    P->d_hist = reinterpret_cast<uint32_t*>(P->d_zero + 8);
    P->d_ohist = P->d_hist + (size_t)nsel * 4096;
    if (P->pk_direct) P->d_pk = reinterpret_cast<uint32_t*>(P->d_zero + pk_off);
    if (P->tail_esz && !P->pk_direct && (rc = dalloc(&P->d_pkb, (size_t)((B * P->tail_esz + 15) / 16) * 4)))
      return fail(rc);
    if ((rc = dalloc(&P->d_key_index, (size_t)P->Lg))) return fail(rc);
    std::vector<int> kidx(P->Lg, -1);
    for (int i = 0; i < nsel; ++i) kidx[P->sel_slots_h[i] - lrank * P->Lg] = i;
    if ((rc = upload(P->d_key_index, kidx.data(), P->Lg * sizeof(int)))) return fail(rc);
    if (cudaMemset(P->d_zero, 0, (size_t)P->nzero * sizeof(int)) != cudaSuccess) {
      g_last_cuda_error = (int)cudaGetLastError();
      return fail(CUSFFT_CUDA);
    }
  }
  if ((rc = dalloc(&P->d_hits, (size_t)P->max_hits))) return fail(rc);
  if ((rc = dalloc(&P->d_hit_vals, (size_t)P->max_hits))) return fail(rc);
  if ((rc = dalloc(&P->d_hit_keys, (size_t)P->max_hits))) return fail(rc);
  if (q.debug && (rc = dalloc(&P->d_per_loop, (size_t)P->max_hits * L))) return fail(rc);
  if ((rc = upload(P->d_slots, P->slots_h.data(), L * sizeof(SlotParam)))) return fail(rc);
  if ((rc = upload(P->d_loc_sigma, loc_sig.data(), P->Lloc * sizeof(uint32_t)))) return fail(rc);
  if (cudaMemset(P->d_records, 0, (size_t)L * P->lay.rec_bytes) != cudaSuccess) {
    g_last_cuda_error = (int)cudaGetLastError();
    return fail(CUSFFT_CUDA);
  }
  cudaError_t ae = set_fft_attrs();
  auto attr = [&](cudaError_t e) {
    if (e != cudaSuccess && ae == cudaSuccess) ae = e;
  };
  attr(set_dyn_smem(k_select1, smem_optin, smem_optin));
  attr(set_dyn_smem(k_select_cluster, 200 * 1024, smem_optin));
  attr(set_dyn_smem(k_select_sort, 210 * 1024, smem_optin));
  attr(set_dyn_smem(k_fft2_select<64, 16>, fft2sel_smem_bytes<64, 16>(), smem_optin));
  attr(set_dyn_smem(k_fft2_select<128, 16>, fft2sel_smem_bytes<128, 16>(), smem_optin));
  attr(set_dyn_smem(k_fft2_select<128, 32>, fft2sel_smem_bytes<128, 32>(), smem_optin));
  attr(set_dyn_smem(k_vote, smem_optin, smem_optin));
  attr(set_dyn_smem(k_output, smem_optin, smem_optin));
  // (the per-function limits are raised to the device maximum, never lowered to this plan's
  // need: plans of other shapes share the kernels)
  if (P->tail_esz) attr(set_dyn_smem(tail_kernel(P->tail_esz, L, P->Lloc), smem_optin, smem_optin));
  if (P->tail_esz && q.shard_mode == 2) attr(set_dyn_smem(tail_vote_kernel(P->tail_esz, P->Lloc), smem_optin, smem_optin));
  if (ae != cudaSuccess) {
    g_last_cuda_error = (int)ae;
    return fail(CUSFFT_CUDA);
  }
  if (P->tail_esz) {  // a warp per (enumerated loop, J) unit; CTAs up to the resident limit
    int occ = 0;
    const cudaError_t oe =
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, tail_kernel(P->tail_esz, L, P->Lloc), kTailNT, P->tail_smem);
    if (oe != cudaSuccess || occ < 1) occ = 1;
    cudaGetLastError();
    const int nenum = (P->T > (P->Lloc + 1) / 2) ? P->Lloc / 2 : P->Lloc - P->T + 1;
    const int64_t units = (int64_t)nenum * (q.cutoff_mode == CUSFFT_CUTOFF_THRESHOLD ? B : P->num);
    const int64_t ctas = (units + kTailNT / 32 - 1) / (kTailNT / 32);
    P->tail_grid = (int)std::max<int64_t>(1, std::min<int64_t>(ctas, (int64_t)P->sms * occ));
  }
  for (int f = 0; f < P->nfilt; ++f)
    if ((rc = build_filter(P, P->filt[f]))) return fail(rc);
  k_twiddles<<<(int)((B + 255) / 256), 256, 0, P->stream>>>(P->d_tw, (int)B);
  if (cudaGetLastError() != cudaSuccess) return fail(CUSFFT_CUDA);
  {  // the estimation's phase e^{-2 pi i m / n} as a product of two tables (m's high / low bits)
    const int log2n = ilog2(n);
    P->plo = (log2n + 1) / 2;
    const int nhi = (int)(n >> P->plo), nlo = 1 << P->plo;
    if ((rc = dalloc(&P->d_ph_hi, (size_t)nhi)) || (rc = dalloc(&P->d_ph_lo, (size_t)nlo))) return fail(rc);
    k_phase_table<<<(nhi + 255) / 256, 256, 0, P->stream>>>(P->d_ph_hi, nhi, P->plo, log2n);
    k_phase_table<<<(nlo + 255) / 256, 256, 0, P->stream>>>(P->d_ph_lo, nlo, 0, log2n);
    if (cudaGetLastError() != cudaSuccess) return fail(CUSFFT_CUDA);
  }
  // ---- distinct 32-B sectors (2 complex samples) of x this rank gathers (the fold's DRAM floor)
  {
    std::vector<uint64_t> bits((size_t)((n / 2 + 63) / 64), 0ull);
    const uint32_t nm = (uint32_t)(n - 1);
    for (int sl = 0; sl < P->Lg; ++sl) {
      const SlotParam& sp = P->slots_h[(size_t)lrank * P->Lg + sl];
      const int w = P->filt[P->filt_of_local(sl)].w;
      for (int i = 0; i < w; ++i) {
        const uint32_t pos = (sp.sigma * (uint32_t)i + sp.tau) & nm;
        if (pos - P->xlo >= P->xspan) continue;
        const uint32_t sec = pos >> 1;
        bits[sec >> 6] |= 1ull << (sec & 63);
      }
    }
    int64_t cnt = 0;
    for (uint64_t b : bits) cnt += __builtin_popcountll(b);
    P->sectors = cnt;
  }
  // ---- staged gather: every (local slot, tap) gather sorted by address at plan time, in
  // groups of consecutive slots whose staging fits L2 (one group when all of it does)
  {
    int rmax = 0;
    int64_t total = 0, rows_all = 0;
    for (int sl = 0; sl < P->Lg; ++sl) {
      rmax = std::max(rmax, P->filt[P->filt_of_local(sl)].R);
      total += P->filt[P->filt_of_local(sl)].w;
      rows_all += P->filt[P->filt_of_local(sl)].R;
    }
    P->stage_total = total;
    const int64_t cap_rows = ((int64_t)64 << 20) / (B * 16);  // staging of one group <= 64 MB
    int gs = rows_all <= cap_rows ? P->Lg : (int)std::max<int64_t>(1, cap_rows / std::max(1, rmax));
    bool forced = false;
    if (const char* e = std::getenv("CUSFFT_STAGE_GROUP")) {  // tests / A/B: force the group size
      gs = std::max(1, std::atoi(e));
      forced = true;
    }
    // several groups never straddle the location / estimation boundary (one filter and one
    // branch each)
    P->grp_s.clear();
    for (int a = 0; a < P->Lg;) {
      const int lim = (gs >= P->Lg) ? P->Lg : a < P->nloc_local ? P->nloc_local : P->Lg;
      P->grp_s.push_back(a);
      a = std::min(lim, a + gs);
    }
    P->grp_s.push_back(P->Lg);
    const int ng = (int)P->grp_s.size() - 1;
    // rows: relative to the group (one shared buffer, groups staged one after the other) unless
    // the staging of all loops fits, when every group keeps its own rows (groups may overlap)
    P->grp_abs = rows_all <= cap_rows;
    P->row0_h.assign((size_t)P->Lg + 1, 0u);
    int64_t rows_max = 0;
    int gmax = 1;
    {
      int64_t rows = 0;
      for (int g = 0; g < ng; ++g) {
        if (!P->grp_abs) rows = 0;
        for (int sl = P->grp_s[g]; sl < P->grp_s[g + 1]; ++sl) {
          P->row0_h[sl] = (uint32_t)rows;
          rows += P->filt[P->filt_of_local(sl)].R;
        }
        rows_max = std::max(rows_max, rows);
        gmax = std::max(gmax, P->grp_s[g + 1] - P->grp_s[g]);
      }
    }
    P->row0_h[P->Lg] = (uint32_t)rows_max;
    int ib = 1;
    while ((int64_t(1) << ib) < P->wmax) ++ib;
    int sb = 0;
    while ((1 << sb) < gmax) ++sb;
    P->stage_ibits = ib;
    const int64_t staging_bytes = rows_max * B * 16;
    // the staging buffer must be (mostly) L2-resident between the two phases, phase 2
    // streams a CTA's R rows (4 KB each) into shared memory, and the schedule word must
    // hold (slot in group, tap); signal-sharded plans gather only their slice (direct path)
    // (signal-sharded plans stage only their own samples: the other entries stay the zeros the
    // staging buffer gets at plan time, so their groups must keep their own rows)
    P->staged = P->fused1 && (!P->xshard || P->grp_abs || ng == 1) && q.gather == 0 &&
                (forced || staging_bytes <= (int64_t)64 << 20) && rmax <= 48 &&
                ib + sb <= 32 && total < (int64_t)1 << 31;
    if (P->staged) {
      const uint32_t nm = (uint32_t)(n - 1);
      std::vector<uint32_t> code;
      code.reserve((size_t)total);
      P->grp_off.assign((size_t)ng + 1, 0);
      std::vector<uint64_t> ev;
      for (int g = 0; g < ng; ++g) {
        ev.clear();
        for (int sl = P->grp_s[g]; sl < P->grp_s[g + 1]; ++sl) {
          const SlotParam& sp = P->slots_h[(size_t)lrank * P->Lg + sl];
          const int w = P->filt[P->filt_of_local(sl)].w;
          const uint64_t sg = (uint64_t)(sl - P->grp_s[g]) << ib;
          for (int i = 0; i < w; ++i) {
            const uint32_t pos = (sp.sigma * (uint32_t)i + sp.tau) & nm;
            if (pos - P->xlo >= P->xspan) continue;  // signal-sharded: another rank's sample
            ev.push_back(((uint64_t)pos << 32) | sg | (uint64_t)i);
          }
        }
        std::sort(ev.begin(), ev.end());
        const int64_t o = P->grp_off[g];
        for (size_t j = 0; j < ev.size(); ++j) code.push_back((uint32_t)(ev[j] & 0xFFFFFFFFull));
        P->grp_off[g + 1] = o + (int64_t)ev.size();
      }
      if ((rc = dalloc(&P->d_code, code.size()))) return fail(rc);
      if ((rc = upload(P->d_code, code.data(), code.size() * sizeof(uint32_t)))) return fail(rc);
      if ((rc = dalloc(&P->d_row0, (size_t)P->Lg))) return fail(rc);
      if ((rc = upload(P->d_row0, P->row0_h.data(), (size_t)P->Lg * sizeof(uint32_t)))) return fail(rc);
      if ((rc = dalloc(&P->d_staging, (size_t)(rows_max * B)))) return fail(rc);
      if (P->xshard && cudaMemset(P->d_staging, 0, (size_t)(rows_max * B) * sizeof(double2)) != cudaSuccess) {
        g_last_cuda_error = (int)cudaGetLastError();  // (entries of other ranks' samples stay 0)
        return fail(CUSFFT_CUDA);
      }
      // one resident wave of phase-1 CTAs (grid-stride loop), at most 4 per SM: with one gather in
      // flight per thread (schedule words prefetched) that is 1024 per SM, measured best
      // (profiles/r02_stage_ab.md; dynamic chunking of the last quarter measured slower)
      int occ = 0;
      if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_stage_packed<kStageU>, 256, 0) != cudaSuccess || occ < 1) occ = 4;
      cudaGetLastError();
      const int per = 256 * kStageU;
      int cps = std::min(occ, 4);
      int64_t gtot = 0;
      for (int g = 0; g < ng; ++g) gtot = std::max(gtot, P->grp_off[g + 1] - P->grp_off[g]);
      // sparse sweeps (fewer than 3 gathers per KB of x, e.g. C4's 4-loop groups: 1.5) are faster
      // with half the requests in flight (2 CTAs per SM: C4 304.5 -> 295.3 us); denser ones (C3: 7,
      // C5 k = 1000: 25, k = 4096: 50 per KB) with 4 (profiles/r02_stage_ab.md)
      if ((double)gtot * 1024.0 / ((double)P->xspan * 16.0) < 3.0) cps = std::min(cps, 2);
      if (const char* e = std::getenv("CUSFFT_STAGE_CPS")) cps = std::max(1, std::min(occ, std::atoi(e)));  // A/B (measurement)
      P->stage_grid = (int)std::max<int64_t>(1, std::min<int64_t>((gtot + per - 1) / per, (int64_t)P->sms * cps));
      // Persisting-L2 set-aside for the staging buffer: the staging stores carry evict_last
      // (= persisting) and the x loads evict_first; C3 is 3 us slower without it
      // (profiles/r02_stage_ab.md).  Device-wide and optional (params.l2_persist).
      int maxp = 0;
      cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev);
      const size_t win = std::min<size_t>((size_t)staging_bytes, (size_t)maxp);
      if (q.l2_persist && win > 0) {
        setaside_acquire(dev, win);
        P->setaside = true;
      }
    }
  }
  if (q.gather == 2 && !P->staged) {  // the remap ablation: one chunk buffer and stream per concurrent loop
    P->remap = true;
    const int nrm = std::min(P->Lg, 32);  // GK110's 32 concurrent kernels (L351)
    if ((rc = dalloc(&P->d_remap, (size_t)nrm * B))) return fail(rc);
    P->rm_st.assign((size_t)nrm, nullptr);
    P->rm_ev.assign((size_t)nrm + 1, nullptr);
    for (auto& st : P->rm_st)
      if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) != cudaSuccess) {
        g_last_cuda_error = (int)cudaGetLastError();
        return fail(CUSFFT_CUDA);
      }
    for (auto& e : P->rm_ev)
      if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) {
        g_last_cuda_error = (int)cudaGetLastError();
        return fail(CUSFFT_CUDA);
      }
  }
  if (q.shard_mode == 2) {  // two all-gathers: candidate records, then per-loop estimates (exchange.cuh)
    P->mode2 = true;
    P->cmax = (P->Lloc + world - 1) / world;
    P->crec_bytes = P->lay.rec_bytes - P->lay.off_bitmap;
    if (set_dyn_smem(k_rank_est, smem_optin, smem_optin) != cudaSuccess) {  // k_rank_est stages the hit list
      g_last_cuda_error = (int)cudaGetLastError();
      return fail(CUSFFT_CUDA);
    }
    if ((rc = dalloc(&P->d_cand, (size_t)(world * P->cmax * P->crec_bytes)))) return fail(rc);
    if ((rc = dalloc(&P->d_x2, (size_t)world * P->max_hits * P->Lg))) return fail(rc);
    if ((rc = dalloc(&P->d_hits2, (size_t)P->max_hits))) return fail(rc);
  }
  if (nccl_id) {  // the library-owned exchange (a world of 1 is allowed: a one-rank communicator)
    ncclUniqueId id;
    std::memcpy(&id, nccl_id, sizeof(id));
    const ncclResult_t nr = api->CommInitRank(&P->comm, world, id, rank);
    if (nr != ncclSuccess) {
      g_last_nccl_error = (int)nr;
      P->comm = nullptr;
      return fail(CUSFFT_NCCL);
    }
  }
  if (cudaStreamSynchronize(P->stream) != cudaSuccess) {
    g_last_cuda_error = (int)cudaGetLastError();
    return fail(CUSFFT_CUDA);
  }
  *out = P;
  return CUSFFT_SUCCESS;
}

// Stage events.  timing 1: between direct launches (every boundary);
// timing 2: event-record nodes of the whole-transform graph around phase 1
// and at the end (ev[0], ev[7], ev[6]), so the gather is timed in the graph
// the bench times.
inline void mark(cusfft_plan_t P, int i) {
  if (P->timing == 1) cudaEventRecord(P->ev[i], P->stream);
  if (P->timing == 2 && (i == 0 || i == 6 || i == 7)) cudaEventRecordWithFlags(P->ev[i], P->stream, cudaEventRecordExternal);
}

// ---------------------------------------------------------------------------
// Launch helpers
// ---------------------------------------------------------------------------
// Staged fold, phase 1: every gather of this rank in address order, each
// sample stored at its phase-2 position.  Zeroes the per-execution block.
int launch_stage1(cusfft_plan_t P, const double2* x, cudaStream_t st, int g = 0) {
  const int s0 = P->grp_s[(size_t)g], s1 = P->grp_s[(size_t)g + 1];
  const int64_t o = P->grp_off[(size_t)g];
  const ZeroArgs z = g == 0 ? ZeroArgs{P->d_zero, P->nzero} : ZeroArgs{nullptr, 0};
  // (signal-sharded: x holds samples [xlo, xlo + xspan); the kernel indexes by the absolute position)
  StagePackArgs a{x - P->xlo, P->d_code + o, P->d_staging, P->d_slots + (size_t)P->lrank * P->Lg + s0, P->d_row0 + s0,
                  (int)(P->grp_off[(size_t)g + 1] - o), s1 - s0, P->stage_ibits, ilog2(P->B), P->logB2, P->logB1,
                  ilog2(256 / P->B1), (uint32_t)(P->n - 1), z,
                  // staging rows to prefetch into L2: the whole buffer, by the first group (later
                  // groups of a shared buffer find the lines the previous group used)
                  g == 0 ? (int)P->row0_h[(size_t)P->Lg] : 0};
  CK(launch_k(k_stage_packed<kStageU>, dim3(P->stage_grid), dim3(256), 0, st, P->cur_prio, a));
  return CUSFFT_SUCCESS;
}

template <int B1T>
cudaError_t launch_p2_t(cusfft_plan_t P, const Filter& F, const double2* staging, double2* u, double2* v, int nslots,
                        ZeroArgs z, cudaStream_t st) {
  static thread_local bool attr_set = false;  // one flag per B1T instantiation
  if (!attr_set) {  // static + dynamic smem may exceed the 48 KB default
    cudaFuncSetAttribute(k_fold_fft1_tma<B1T, 8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    cudaFuncSetAttribute(k_fold_fft1_tma<B1T, 16>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    attr_set = true;
  }
  if (P->p2_ms && F.R <= 16) {  // multi-slot form (k_fold_fft1_ms)
    // R <= 8: 8 slots per CTA, 4 in flight.  8 < R <= 16: 8 slots per CTA with 2 in flight
    // (one CTA per SM), or 4 slots per CTA with 1 in flight (two CTAs per SM) for ranges of at
    // most 4 slots or B <= 16384 (C4: 333 -> 325 us, C5 k = 1000: 62.1 -> 57.5 us; B = 32768
    // ranges of 8 slots, C5 k = 4096, are faster with 8: profiles/r02_stage_ab.md)
    static thread_local bool ms_attr = false;
    if (!ms_attr) {
      cudaFuncSetAttribute(k_fold_fft1_ms<B1T, 8, 4, 8>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           fold_ms_smem_bytes<B1T, 8, 4, 8>());
      cudaFuncSetAttribute(k_fold_fft1_ms<B1T, 8, 2, 16>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           fold_ms_smem_bytes<B1T, 8, 2, 16>());
      cudaFuncSetAttribute(k_fold_fft1_ms<B1T, 4, 1, 16>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           fold_ms_smem_bytes<B1T, 4, 1, 16>());
      ms_attr = true;
    }
    auto kern = k_fold_fft1_ms<B1T, 8, 4, 8>;
    int nsm = 8, smem = fold_ms_smem_bytes<B1T, 8, 4, 8>();
    if (F.R > 8 && (nslots <= 4 || P->B <= 16384)) {
      kern = k_fold_fft1_ms<B1T, 4, 1, 16>;
      nsm = 4;
      smem = fold_ms_smem_bytes<B1T, 4, 1, 16>();
    } else if (F.R > 8) {
      kern = k_fold_fft1_ms<B1T, 8, 2, 16>;
      smem = fold_ms_smem_bytes<B1T, 8, 2, 16>();
    }
    dim3 grid((unsigned)(P->B / 256), (unsigned)((nslots + nsm - 1) / nsm));
    return launch_k(kern, grid, dim3(256), (size_t)smem, st, P->cur_prio, staging, (const double*)F.d_taps_perm,
                    P->prm.debug ? u : nullptr, v, (const double2*)P->d_tw, (int)P->B, P->B2, F.w, F.R, nslots, z);
  }
  // spc slots per CTA (their taps loaded once), double-buffered rows while two fit in shared memory
  const int spc = (2 * F.R * 4096 <= 160 * 1024) ? std::min(P->p2_spc, nslots) : 1;
  const size_t smem = (size_t)(spc > 1 ? 2 : 1) * F.R * 4096;
  dim3 grid((unsigned)(P->B / 256), (unsigned)((nslots + spc - 1) / spc));
  auto kern = F.R <= 8 ? k_fold_fft1_tma<B1T, 8> : k_fold_fft1_tma<B1T, 16>;
  return launch_k(kern, grid, dim3(256), smem, st, P->cur_prio, staging,
                  (const double*)F.d_taps_perm, P->prm.debug ? u : nullptr, v, (const double2*)P->d_tw, (int)P->B,
                  P->B2, F.w, F.R, nslots, spc, z);
}

template <int B1T>
cudaError_t launch_direct_t(cusfft_plan_t P, const Filter& F, const double2* x, const SlotParam* sp, double2* u,
                            double2* v, int nslots, ZeroArgs z, cudaStream_t st) {
  dim3 grid((unsigned)(P->B / 256), (unsigned)nslots);
  return launch_k(k_fold_fft1<B1T, 8>, grid, dim3(256), 0, st, P->cur_prio, x, (const double*)F.d_taps_perm, sp, u, v,
                  (const double2*)P->d_tw, (int)P->B, P->B2, F.w, F.R, (uint32_t)(P->n - 1), P->xlo, P->xspan, z);
}

// Steps 1+2 as the paper's asynchronous data layout transformation (gather 2,
// PAPER.md:L345-L351, Fig. 4): per loop and chunk of B taps a remapping kernel
// (A'[j] = x[index]) and an execution kernel (u += g A'); loop s on stream
// s mod nrm, the streams forked from and joined back to st.
int launch_remap(cusfft_plan_t P, const double2* x, int s0, int s1, cudaStream_t st, bool zero_block) {
  const int B = (int)P->B;
  const int nrm = (int)P->rm_st.size();
  if (zero_block) CK(cudaMemsetAsync(P->d_zero, 0, (size_t)P->nzero * sizeof(int), st));
  CK(cudaEventRecord(P->rm_ev[0], st));
  for (int i = 0; i < nrm; ++i) CK(cudaStreamWaitEvent(P->rm_st[(size_t)i], P->rm_ev[0], 0));
  const dim3 grid((unsigned)((B + 255) / 256)), blk(256);
  for (int s = s0; s < s1; ++s) {
    const int i = (s - s0) % nrm;
    cudaStream_t rs = P->rm_st[(size_t)i];
    double2* ap = P->d_remap + (size_t)i * B;
    const Filter& F = P->filt[P->filt_of_local(s)];
    const SlotParam& sp = P->slots_h[(size_t)P->lrank * P->Lg + s];
    double2* u = P->d_u + (size_t)s * B;
    for (int rr = 0; rr < F.R; ++rr) {
      k_remap<<<grid, blk, 0, rs>>>(x, ap, sp.sigma, sp.tau, rr * B, B, F.w, (uint32_t)(P->n - 1));
      k_remap_exec<<<grid, blk, 0, rs>>>(ap, (const double*)F.d_taps, u, rr * B, B, F.w);
    }
  }
  CK(cudaGetLastError());
  for (int i = 0; i < nrm; ++i) {
    CK(cudaEventRecord(P->rm_ev[(size_t)i + 1], P->rm_st[(size_t)i]));
    CK(cudaStreamWaitEvent(st, P->rm_ev[(size_t)i + 1], 0));
  }
  return CUSFFT_SUCCESS;
}

// Steps 1+2 (and the fused FFT pass 1) for local slots [s0, s1), all of one
// filter: phase 2 of the staged fold, or the direct gather.
int launch_fold_range(cusfft_plan_t P, const double2* x, int s0, int s1, cudaStream_t st, bool zero_block) {
  if (s1 <= s0) return CUSFFT_SUCCESS;
  const int64_t B = P->B;
  const Filter& F = P->filt[P->filt_of_local(s0)];
  const SlotParam* sp = P->d_slots + (size_t)P->lrank * P->Lg + s0;
  double2* u = P->d_u + (size_t)s0 * B;
  double2* v = P->d_v ? P->d_v + (size_t)s0 * B : nullptr;
  const ZeroArgs z{zero_block ? P->d_zero : nullptr, zero_block ? P->nzero : 0};
  cudaError_t e = cudaErrorInvalidValue;
  if (P->staged) {
    const double2* stg = P->d_staging + (size_t)P->row0_h[s0] * B;
    switch (P->B1) {
      case 64: e = launch_p2_t<64>(P, F, stg, u, v, s1 - s0, z, st); break;
      case 128: e = launch_p2_t<128>(P, F, stg, u, v, s1 - s0, z, st); break;
      case 256: e = launch_p2_t<256>(P, F, stg, u, v, s1 - s0, z, st); break;
    }
  } else if (P->fused1) {
    switch (P->B1) {
      case 64: e = launch_direct_t<64>(P, F, x, sp, u, v, s1 - s0, z, st); break;
      case 128: e = launch_direct_t<128>(P, F, x, sp, u, v, s1 - s0, z, st); break;
      case 256: e = launch_direct_t<256>(P, F, x, sp, u, v, s1 - s0, z, st); break;
    }
  } else if (P->remap) {
    return launch_remap(P, x, s0, s1, st, zero_block);
  } else {
    dim3 grid((unsigned)((B + 255) / 256), (unsigned)(s1 - s0));
    e = launch_k(k_fold<16>, grid, dim3(256), 0, st, P->cur_prio, x, (const double*)F.d_taps, sp, u, (int)B, F.w,
                 F.R, (uint32_t)(P->n - 1), P->xlo, P->xspan, z);
  }
  CK(e);
  return CUSFFT_SUCCESS;
}

// Step 3 (remaining FFT passes, cutoff keys) for local slots [s0, s1).
int launch_bfft(cusfft_plan_t P, int s0, int s1, cudaStream_t st) {
  if (s1 <= s0) return CUSFFT_SUCCESS;
  const int B = (int)P->B;
  const int ns = s1 - s0;
  double2* rec = reinterpret_cast<double2*>(P->d_records + ((int64_t)P->lrank * P->Lg + s0) * P->lay.rec_bytes);
  const int64_t rec_e = P->lay.rec_bytes / 16;
  // signal-sharded: the spectra are partial here, keys come after the all-reduce (launch_keys)
  const int* kidx = (P->sel_slots_h.empty() || P->xshard) ? nullptr : P->d_key_index + s0;
  if (P->B1 > 1) {
    if (!P->fused1) {  // pass 1: B1-point FFTs over columns c (stride B2), twiddle e^{-2 pi i c k1 / B}
      FftPassArgs a1{P->d_u + (size_t)s0 * B, P->d_v + (size_t)s0 * B, P->d_tw, B, P->logB2, ns * P->B2, B, B, 1,
                     P->B2, 1, P->B2, 1, nullptr, nullptr, nullptr};
      CK(launch_fft(P->B1, a1, st, P->cur_prio));
    }
    // pass 2: B2-point FFTs of contiguous rows k1, out to u^[k1 + B1 k2] (+ cutoff keys)
    FftPassArgs a2{P->d_v + (size_t)s0 * B, rec, P->d_tw, B, P->logB1, ns * P->B1, B, rec_e, P->B2, 1, 1, P->B1, 0,
                   kidx, P->d_keys, P->d_hist};
    CK(launch_fft(P->B2, a2, st, P->cur_prio));
  } else {
    FftPassArgs a{P->d_u + (size_t)s0 * B, rec, P->d_tw, B, 0, ns, B, rec_e, 0, 1, 0, 1, 0, kidx, P->d_keys,
                  P->d_hist};
    CK(launch_fft(P->B2, a, st, P->cur_prio));
  }
  return CUSFFT_SUCCESS;
}

// Step 4 for this rank's location slots.
SelArgs make_sel_args(cusfft_plan_t P) {
  SelArgs sa{};
  for (size_t i = 0; i < P->sel_slots_h.size(); ++i)
    sa.recs[i] = P->d_records + (int64_t)P->sel_slots_h[i] * P->lay.rec_bytes;
  sa.lay = P->lay;
  sa.B = (int)P->B;
  sa.num = P->num;
  sa.keys = P->d_keys;
  sa.hist0 = P->d_hist;
  sa.status = P->d_flags + 1;
  sa.pk = P->d_pk;
  sa.pk_esz = P->tail_esz;
  if (P->mode2)  // this rank's location slots are its first local slots, in order
    for (size_t i = 0; i < P->sel_slots_h.size(); ++i)
      sa.cout[i] = P->d_cand + ((int64_t)P->rank * P->cmax + (int64_t)i) * P->crec_bytes;
  sa.threshold_mode = P->prm.cutoff_mode == CUSFFT_CUTOFF_THRESHOLD ? 1 : 0;
  {
    const double th = P->prm.cutoff_threshold;
    uint64_t bits;
    std::memcpy(&bits, &th, 8);
    sa.thr_key = bits;
  }
  return sa;
}

int launch_select(cusfft_plan_t P, cudaStream_t st) {
  if (P->sel_slots_h.empty()) return CUSFFT_SUCCESS;
  const SelArgs sa = make_sel_args(P);
  const int nsel = (int)P->sel_slots_h.size();
  if (P->prm.cutoff_mode == CUSFFT_CUTOFF_SORT) {
    const int smem = (int)P->B * 12 + (int)((P->B + 31) / 32) * 4;
    CK(launch_k(k_select_sort, dim3(nsel), dim3(1024), smem, st, P->cur_prio, sa));
    return CUSFFT_SUCCESS;
  }
  if (P->sel_cluster) {
    const int smem = (int)sizeof(SelClusterSmem) + (int)(P->B / kSelCL / 32) * 4;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(nsel * kSelCL));
    cfg.blockDim = dim3(kSelCNT);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[3];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = kSelCL;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[1].val.programmaticStreamSerializationAllowed = g_pdl ? 1 : 0;
    attr[2].id = cudaLaunchAttributePriority;
    attr[2].val.priority = P->cur_prio;
    cfg.attrs = attr;
    cfg.numAttrs = 3;
    CK(cudaLaunchKernelEx(&cfg, k_select_cluster, sa));
    return CUSFFT_SUCCESS;
  }
  CK(launch_k(k_select1, dim3(nsel), dim3(1024), P->select1_smem, st, P->cur_prio, sa));
  return CUSFFT_SUCCESS;
}

// FFT pass 2 + cutoff of the location slots in one cluster kernel
// (k_fft2_select): exact mode, four-step B with B1 = 8 ROWS, the selected
// slots = this rank's location slots [0, nloc_local) in order, shapes with
// compiled instances (B = 8192, 16384, 32768).
bool use_fft2_select(cusfft_plan_t P) {
  // (the location slots' FFT pass 1 must have run inside the fold: fused1)
  if (!P->sel_cluster || P->xshard || P->prm.cutoff_mode != CUSFFT_CUTOFF_EXACT || P->B1 <= 1 || !P->fft2sel ||
      !P->fused1)
    return false;
  const int key = P->B2 * 1000 + P->B1 / kSelCL;
  if (key != 64016 && key != 128016 && key != 128032) return false;
  if ((int)P->sel_slots_h.size() != P->nloc_local) return false;
  for (int i = 0; i < P->nloc_local; ++i)
    if (P->sel_slots_h[(size_t)i] != (int64_t)P->lrank * P->Lg + i) return false;
  return true;
}

template <int M, int ROWS>
cudaError_t launch_f2s_t(cusfft_plan_t P, const Fft2SelArgs& fa, int nsel, cudaStream_t st) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(nsel * kSelCL));
  cfg.blockDim = dim3(kF2SNT);
  cfg.dynamicSmemBytes = (size_t)fft2sel_smem_bytes<M, ROWS>();
  cfg.stream = st;
  cudaLaunchAttribute attr[3];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = kSelCL;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = g_pdl ? 1 : 0;
  attr[2].id = cudaLaunchAttributePriority;
  attr[2].val.priority = P->cur_prio;
  cfg.attrs = attr;
  cfg.numAttrs = 3;
  return cudaLaunchKernelEx(&cfg, k_fft2_select<M, ROWS>, fa);
}

int launch_fft2_select(cusfft_plan_t P, cudaStream_t st) {
  const int nsel = (int)P->sel_slots_h.size();
  if (nsel == 0) return CUSFFT_SUCCESS;
  Fft2SelArgs fa{};
  fa.s = make_sel_args(P);
  for (int i = 0; i < nsel; ++i) fa.v[i] = P->d_v + (size_t)i * P->B;
  fa.tw = P->d_tw;
  fa.B1 = P->B1;
  cudaError_t e = cudaErrorInvalidValue;
  switch (P->B2 * 1000 + P->B1 / kSelCL) {
    case 64016: e = launch_f2s_t<64, 16>(P, fa, nsel, st); break;
    case 128016: e = launch_f2s_t<128, 16>(P, fa, nsel, st); break;
    case 128032: e = launch_f2s_t<128, 32>(P, fa, nsel, st); break;
  }
  CK(e);
  return CUSFFT_SUCCESS;
}

// Cutoff keys from the summed spectra (signal-sharded plans, after the exchange).
int launch_keys(cusfft_plan_t P, cudaStream_t st) {
  if (P->sel_slots_h.empty()) return CUSFFT_SUCCESS;
  KeysArgs ka{};
  for (size_t i = 0; i < P->sel_slots_h.size(); ++i)
    ka.rec[i] = reinterpret_cast<const double2*>(P->d_records + (int64_t)P->sel_slots_h[i] * P->lay.rec_bytes);
  ka.keys = P->d_keys;
  ka.hist = P->d_hist;
  ka.B = (int)P->B;
  const int gx = (int)std::max<int64_t>(1, std::min<int64_t>(P->B / 1024, 64));
  CK(launch_k(k_keys, dim3(gx, (unsigned)P->sel_slots_h.size()), dim3(256), 0, st, P->cur_prio, ka));
  return CUSFFT_SUCCESS;
}

VoteArgs make_vote_args(cusfft_plan_t P) {
  VoteArgs va{};
  for (int q = 0; q < P->Lloc; ++q) {
    const uint8_t* rec = P->d_records + (int64_t)P->loc_slots_h[q] * P->lay.rec_bytes;
    va.bmp[q] = reinterpret_cast<const uint32_t*>(rec + P->lay.off_bitmap);
    va.Jp[q] = reinterpret_cast<const int*>(rec + P->lay.off_J);
    va.cntp[q] = reinterpret_cast<const int*>(rec + P->lay.off_cnt);
    if (P->mode2) {  // the gathered candidate record: rank g = slot / Lg, its location slot i = slot mod Lg
      const int64_t s = P->loc_slots_h[q];
      const uint8_t* c = P->d_cand + ((s / P->Lg) * P->cmax + s % P->Lg) * P->crec_bytes;
      va.bmp[q] = reinterpret_cast<const uint32_t*>(c);
      va.Jp[q] = reinterpret_cast<const int*>(c + (P->lay.off_J - P->lay.off_bitmap));
      va.cntp[q] = reinterpret_cast<const int*>(c + (P->lay.off_cnt - P->lay.off_bitmap));
    }
    va.sig[q] = P->slots_h[P->loc_slots_h[q]].sigma;
    va.aa[q] = P->slots_h[P->loc_slots_h[q]].a;
  }
  va.loc_sigma = P->d_loc_sigma;
  va.Lloc = P->Lloc;
  va.T = P->T;
  va.num = P->num;
  va.B = (int)P->B;
  va.nb = (int)P->nb;
  va.log2nb = P->log2nb;
  va.log2n = ilog2(P->n);
  va.log2B = ilog2(P->B);
  va.nmask = (uint32_t)(P->n - 1);
  va.pairs = P->T > (P->Lloc + 1) / 2 ? 1 : 0;
  va.cnt_fixed = P->prm.cutoff_mode == CUSFFT_CUTOFF_THRESHOLD ? 0 : 1;
  va.hits = P->d_hits;
  va.hit_count = reinterpret_cast<unsigned*>(P->d_flags);
  va.max_hits = P->max_hits;
  va.pk = P->d_pk ? P->d_pk : P->d_pkb;
  return va;
}

EstArgs make_est_args(cusfft_plan_t P) {
  EstArgs ea{};
  ea.records = P->d_records;
  ea.lay = P->lay;
  ea.slots = P->d_slots;
  ea.L = P->L;
  ea.ginv = P->filt[0].d_ginv;
  ea.ginv_est = P->filt[P->nfilt - 1].d_ginv;
  ea.ghat_split = P->nfilt > 1 ? P->Lloc : P->L;
  ea.ph_hi = P->d_ph_hi;
  ea.ph_lo = P->d_ph_lo;
  ea.plo = P->plo;
  ea.hits = P->d_hits;
  ea.hit_count = reinterpret_cast<const unsigned*>(P->d_flags);
  ea.max_hits = P->max_hits;
  ea.nmask = (uint32_t)(P->n - 1);
  ea.log2nb = P->log2nb;
  ea.nb = (int)P->nb;
  ea.B = (int)P->B;
  ea.n = (double)P->n;
  ea.hit_vals = P->d_hit_vals;
  ea.hit_keys = P->d_hit_keys;
  ea.per_loop = P->d_per_loop;
  ea.out_hist = P->d_ohist;
  return ea;
}

// The vote table from the cutoff bitmaps (fused-tail plans whose cutoff does not OR into it).
int launch_pk_build(cusfft_plan_t P, cudaStream_t st) {
  if (!P->d_pkb) return CUSFFT_SUCCESS;
  const VoteArgs va = make_vote_args(P);
  const dim3 grid((unsigned)((P->B + 255) / 256));
  cudaError_t e;
  if (P->tail_esz == 1)
    e = launch_k(k_pk_build<uint8_t>, grid, dim3(256), 0, st, P->cur_prio, va, reinterpret_cast<uint8_t*>(P->d_pkb));
  else if (P->tail_esz == 2)
    e = launch_k(k_pk_build<uint16_t>, grid, dim3(256), 0, st, P->cur_prio, va, reinterpret_cast<uint16_t*>(P->d_pkb));
  else
    e = launch_k(k_pk_build<uint32_t>, grid, dim3(256), 0, st, P->cur_prio, va, P->d_pkb);
  CK(e);
  g_pdl = P->timing != 1;
  return CUSFFT_SUCCESS;
}

// Steps 5 + 6 in one kernel (tail.cuh).
int launch_tail(cusfft_plan_t P, cudaStream_t st) {
  TRY(launch_pk_build(P, st));
  TailArgs ta{};
  ta.v = make_vote_args(P);
  ta.e = make_est_args(P);
  ta.q_off = P->tail_qoff;
  CK(launch_k(tail_kernel(P->tail_esz, P->L, P->Lloc), dim3((unsigned)P->tail_grid), dim3(kTailNT),
              (size_t)P->tail_smem, st, P->cur_prio, ta));
  return CUSFFT_SUCCESS;
}

// Steps 5-6 (the fused k_tail, or the chain k_vote -> k_estimate* for plans
// whose vote table does not fit shared memory) and the output (stage limits 4..6).
int launch_after_cutoff(cusfft_plan_t P, int64_t* locs, double2* vals, cudaStream_t st) {
  if (P->stage_limit < 4) return CUSFFT_SUCCESS;
  if (P->tail_esz) {
    TRY(launch_tail(P, st));
    mark(P, 4);
    mark(P, 5);
  } else {
    CK(launch_k(k_vote, dim3(P->vote_grid), dim3(256), P->vote_smem, st, P->cur_prio, make_vote_args(P)));
    mark(P, 4);
    if (P->stage_limit < 5) return CUSFFT_SUCCESS;
    const EstArgs ea = make_est_args(P);
    g_pdl = P->timing != 1;
    if (P->L <= 8)
      CK(launch_k(k_estimate_seg<8>, dim3(P->est_grid), dim3(256), 0, st, P->cur_prio, ea));
    else if (P->L <= 16)
      CK(launch_k(k_estimate_seg<16>, dim3(P->est_grid), dim3(256), 0, st, P->cur_prio, ea));
    else
      CK(launch_k(k_estimate, dim3(P->est_grid), dim3(256), 0, st, P->cur_prio, ea));
    mark(P, 5);
  }
  if (P->stage_limit < 6) return CUSFFT_SUCCESS;
  g_pdl = P->timing != 1;
  CK(launch_k(k_output, dim3(1), dim3(1024), P->output_smem, st, P->cur_prio, (const int*)P->d_hits,
              reinterpret_cast<const unsigned*>(P->d_flags), P->max_hits, (const double2*)P->d_hit_vals,
              (const uint64_t*)P->d_hit_keys, P->d_ohist, (int)P->k, P->kp2, ilog2(P->n), locs, vals,
              P->d_flags + 1));
  mark(P, 6);
  return CUSFFT_SUCCESS;
}

// shard_mode 2, after the candidate all-gather: every rank votes over all
// location loops (k_vote), ranks the hits into ascending order and estimates its
// own loops for every hit into its slice of the estimate buffer (k_rank_est).
int launch_mid(cusfft_plan_t P, cudaStream_t st) {
  if (P->stage_limit < 4) return CUSFFT_SUCCESS;
  if (P->tail_esz) {  // the fused tail's vote, without its estimation
    TRY(launch_pk_build(P, st));
    TailArgs ta{};
    ta.v = make_vote_args(P);
    ta.e = make_est_args(P);
    ta.q_off = P->tail_qoff;
    CK(launch_k(tail_vote_kernel(P->tail_esz, P->Lloc), dim3((unsigned)P->tail_grid), dim3(kTailNT),
                (size_t)P->tail_smem, st, P->cur_prio, ta));
  } else {
    CK(launch_k(k_vote, dim3(P->vote_grid), dim3(256), P->vote_smem, st, P->cur_prio, make_vote_args(P)));
  }
  mark(P, 4);
  if (P->stage_limit < 5) return CUSFFT_SUCCESS;
  g_pdl = P->timing != 1;
  CK(launch_k(k_rank_est, dim3((unsigned)((P->max_hits + kRankC - 1) / kRankC)), dim3(kRankNT),
              (size_t)P->max_hits * 4, st,
              P->cur_prio, make_est_args(P), P->rank * P->Lg, P->Lg, P->d_hits2,
              P->d_x2 + (size_t)P->rank * P->max_hits * P->Lg));
  return CUSFFT_SUCCESS;
}

// shard_mode 2, after the estimate all-gather: medians (k_median) and the output.
int launch_finish2(cusfft_plan_t P, int64_t* locs, double2* vals, cudaStream_t st) {
  if (P->stage_limit < 5) return CUSFFT_SUCCESS;
  const int gx = std::max(1, std::min((P->max_hits + 7) / 8, P->sms * 4));  // a warp per hit
  CK(launch_k(k_median, dim3(gx), dim3(256), 0, st, P->cur_prio, make_est_args(P), (const double2*)P->d_x2,
              P->world, P->Lg));
  mark(P, 5);
  if (P->stage_limit < 6) return CUSFFT_SUCCESS;
  g_pdl = P->timing != 1;
  CK(launch_k(k_output, dim3(1), dim3(1024), P->output_smem, st, P->cur_prio, (const int*)P->d_hits2,
              reinterpret_cast<const unsigned*>(P->d_flags), P->max_hits, (const double2*)P->d_hit_vals,
              (const uint64_t*)P->d_hit_keys, P->d_ohist, (int)P->k, P->kp2, ilog2(P->n), locs, vals,
              P->d_flags + 1));
  mark(P, 6);
  return CUSFFT_SUCCESS;
}

// Steps 1-4 of this rank's loops, one serial chain on P->stream.
int launch_local(cusfft_plan_t P, const double2* x) {
  cudaStream_t st = P->stream;
  mark(P, 0);
  g_pdl = false;  // the first kernel follows arbitrary caller work
  const int nl = P->nloc_local;
  if (P->staged && P->grp_s.size() > 2) {  // stage groups, one after the other through one staging buffer
    for (size_t g = 0; g + 1 < P->grp_s.size(); ++g) {
      TRY(launch_stage1(P, x, st, (int)g));
      g_pdl = P->timing != 1;
      TRY(launch_fold_range(P, x, P->grp_s[g], P->grp_s[g + 1], st, false));
    }
  } else if (P->staged) {
    TRY(launch_stage1(P, x, st));
    mark(P, 7);
    g_pdl = P->timing != 1;
    TRY(launch_fold_range(P, x, 0, nl, st, false));
    TRY(launch_fold_range(P, x, nl, P->Lg, st, false));
  } else {
    TRY(launch_fold_range(P, x, 0, nl, st, true));
    g_pdl = P->timing != 1;
    TRY(launch_fold_range(P, x, nl, P->Lg, st, nl == 0));
  }
  g_pdl = P->timing != 1;
  mark(P, 1);
  if (P->stage_limit < 2) return CUSFFT_SUCCESS;
  const bool f2s = use_fft2_select(P);
  TRY(launch_bfft(P, f2s ? P->nloc_local : 0, P->Lg, st));  // fused: the location slots' pass 2 runs with their cutoff (stage 3)
  mark(P, 2);
  if (P->stage_limit < 3 || P->xshard) return CUSFFT_SUCCESS;  // signal-sharded: cutoff after the all-reduce
  if (f2s)
    TRY(launch_fft2_select(P, st));
  else
    TRY(launch_select(P, st));
  mark(P, 3);
  return CUSFFT_SUCCESS;
}

// Steps 5-6 + output after the exchange (signal-sharded plans: keys + cutoff first).
int launch_finish(cusfft_plan_t P, int64_t* locs, double2* vals) {
  cudaStream_t st = P->stream;
  g_pdl = P->timing != 1;
  if (P->xshard) {
    g_pdl = false;  // follows the all-reduce
    if (P->stage_limit < 3) return CUSFFT_SUCCESS;
    TRY(launch_keys(P, st));
    g_pdl = P->timing != 1;
    TRY(launch_select(P, st));
    mark(P, 3);
  }
  return launch_after_cutoff(P, locs, vals, st);
}

// The library-owned exchange (plans made with an ncclUniqueId): ONE collective
// on the plan's stream, in place on the exchange buffer.
int launch_exchange(cusfft_plan_t P, cudaStream_t st, int which = 0) {
  if (!P->comm) return CUSFFT_SUCCESS;
  const NcclApi* api = nccl_api();
  const size_t per = (size_t)P->Lg * P->lay.rec_bytes;
  ncclResult_t r;
  if (P->mode2) {  // which 1: the candidate records; 2: the per-loop estimates (in place)
    const size_t c = which == 1 ? (size_t)P->cmax * P->crec_bytes : (size_t)P->max_hits * P->Lg * sizeof(double2);
    uint8_t* buf = which == 1 ? P->d_cand : reinterpret_cast<uint8_t*>(P->d_x2);
    r = api->AllGather(buf + (size_t)P->rank * c, buf, c, ncclUint8, P->comm, st);
  } else if (P->xshard)
    r = api->AllReduce(P->d_records, P->d_records, (size_t)P->L * P->lay.rec_bytes / 8, ncclFloat64, ncclSum, P->comm, st);
  else
    r = api->AllGather(P->d_records + (size_t)P->rank * per, P->d_records, per, ncclUint8, P->comm, st);
  if (r != ncclSuccess) {
    g_last_nccl_error = (int)r;
    return CUSFFT_NCCL;
  }
  return CUSFFT_SUCCESS;
}

// shard_mode 2 after Steps 1-4: candidate all-gather, vote + sort + local
// estimates, estimate all-gather, medians + output (exchange.cuh).
int launch_rest2(cusfft_plan_t P, int64_t* locs, double2* vals, cudaStream_t st) {
  g_pdl = false;
  if (P->comm) TRY(launch_exchange(P, st, 1));
  TRY(launch_mid(P, st));
  g_pdl = false;
  if (P->comm) TRY(launch_exchange(P, st, 2));
  return launch_finish2(P, locs, vals, st);
}

// The whole transform as two concurrent branches (graph capture, staged
// plans with location and estimation-only slots on this rank): ONE
// address-ordered phase 1 of every slot, then the location slots' phase 2,
// FFT pass 2 and cutoff on a high-priority stream while the estimation
// slots' phase 2 and FFT pass 2 fill the SMs the latency-bound chain leaves
// idle on a second stream; they join before the exchange / the tail.  The
// estimation branch forks after phase 1 (fork_at 0) or after the location
// slots' phase 2 (fork_at 1: that phase 2 then has the L2 bandwidth alone).
// Stage limits below 6 end the graph early (both branches joined).
int launch_branched(cusfft_plan_t P, const double2* x, int64_t* locs, double2* vals) {
  cudaStream_t a = P->stream, b = P->cap_stream2;
  const int nl = P->nloc_local;
  const int lim = P->stage_limit;
  // two stage groups (location / estimation loops, each with its own staging rows): the
  // estimation loops' phase 1 runs on the second branch, after the location loops' one
  const bool split = P->grp_s.size() == 3;
  auto fork = [&]() -> int {
    CK(cudaEventRecord(P->ev_fork, a));
    CK(cudaStreamWaitEvent(b, P->ev_fork, 0));
    P->cur_prio = P->prio_lo;
    g_pdl = false;
    if (split) {
      TRY(launch_stage1(P, x, b, 1));
      g_pdl = true;
    }
    TRY(launch_fold_range(P, x, nl, P->Lg, b, false));
    g_pdl = true;
    if (lim >= 2) TRY(launch_bfft(P, nl, P->Lg, b));
    CK(cudaEventRecord(P->ev_join, b));
    P->cur_prio = P->prio_hi;
    g_pdl = true;  // the next kernel on a keeps its programmatic edge (the event record adds no node)
    return CUSFFT_SUCCESS;
  };
  P->cur_prio = P->prio_hi;
  g_pdl = false;
  mark(P, 0);
  TRY(launch_stage1(P, x, a));
  if (!split) mark(P, 7);
  if (P->fork_at == 0 || split) TRY(fork());
  g_pdl = true;
  TRY(launch_fold_range(P, x, 0, nl, a, false));
  if (P->fork_at == 1 && !split) TRY(fork());
  const bool f2s = use_fft2_select(P);  // location slots: FFT pass 2 inside the cutoff kernel (stage 3)
  if (lim >= 2 && !f2s) TRY(launch_bfft(P, 0, nl, a));
  if (P->fork_at == 2 && !split) TRY(fork());
  if (f2s && lim >= 3)
    TRY(launch_fft2_select(P, a));
  else if (lim >= 3 && !P->xshard)
    TRY(launch_select(P, a));
  if (P->fork_at == 3 && !split) TRY(fork());
  P->cur_prio = 0;
  CK(cudaStreamWaitEvent(a, P->ev_join, 0));
  g_pdl = false;
  if (lim < 4) return CUSFFT_SUCCESS;
  if (P->mode2) return launch_rest2(P, locs, vals, a);
  if (P->comm) {
    TRY(launch_exchange(P, a));
    return launch_finish(P, locs, vals);
  }
  return launch_after_cutoff(P, locs, vals, a);
}

inline bool use_branches(cusfft_plan_t P) {
  const bool split = P->grp_abs && P->grp_s.size() == 3 && P->grp_s[1] == P->nloc_local;  // phase 1 per branch
  return P->timing != 1 && P->staged && (P->grp_s.size() == 2 || split) && P->nloc_local > 0 &&
         P->nloc_local < P->Lg && !P->xshard;
}

// The plan-owned capture stream, the estimation branch's stream and the fork / join events.
int ensure_streams(cusfft_plan_t P) {
  if (P->cap_stream) return CUSFFT_SUCCESS;
  int lo = 0, hi = 0;
  CK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
  P->prio_lo = lo;
  P->prio_hi = hi;
  CK(cudaStreamCreateWithPriority(&P->cap_stream, cudaStreamNonBlocking, hi));   // location chain
  CK(cudaStreamCreateWithPriority(&P->cap_stream2, cudaStreamNonBlocking, lo));  // estimation folds
  CK(cudaEventCreateWithFlags(&P->ev_fork, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&P->ev_join, cudaEventDisableTiming));
  return CUSFFT_SUCCESS;
}

// Run `body` (which enqueues on P->stream) either directly or through a cached
// CUDA graph captured on a plan-owned stream and launched on the caller's
// stream.  Timing mode launches directly (events between the kernels).
template <class F>
int run_graphed(cusfft_plan_t P, cusfft_plan_s::GraphEntry& g, const void* a, const void* b, const void* c,
                F&& body) {
  if (!P->use_graph || P->timing == 1) return body();
  if (!(g.exec && g.a == a && g.b == b && g.c == c && g.lim == P->stage_limit && g.tmode == P->timing)) {
    if (g.exec) {
      cudaGraphExecDestroy(g.exec);
      g.exec = nullptr;
    }
    TRY(ensure_streams(P));
    CK(cudaStreamBeginCapture(P->cap_stream, cudaStreamCaptureModeThreadLocal));
    cudaStream_t user = P->stream;
    P->stream = P->cap_stream;
    const int rc = body();
    cudaGraph_t graph = nullptr;
    const cudaError_t ce = cudaStreamEndCapture(P->cap_stream, &graph);
    P->stream = user;
    P->cur_prio = 0;
    if (rc != CUSFFT_SUCCESS) {
      if (graph) cudaGraphDestroy(graph);
      return rc;
    }
    CK(ce);
    // node priorities (location branch high, estimation branch low) are honoured only with UseNodePriority
    const cudaError_t ie = cudaGraphInstantiateWithFlags(&g.exec, graph, cudaGraphInstantiateFlagUseNodePriority);
    cudaGraphDestroy(graph);
    CK(ie);
    g.a = a;
    g.b = b;
    g.c = c;
    g.lim = P->stage_limit;
    g.tmode = P->timing;
  }
  CK(cudaGraphLaunch(g.exec, P->stream));
  return CUSFFT_SUCCESS;
}

// The cache entry for a whole-transform graph of (a, b, c) at the current stage limit.
cusfft_plan_s::GraphEntry& full_entry(cusfft_plan_t P, const void* a, const void* b, const void* c) {
  size_t lru = 0;
  for (size_t i = 0; i < P->g_cache.size(); ++i) {
    const auto& g = P->g_cache[i];
    if (g.exec && g.a == a && g.b == b && g.c == c && g.lim == P->stage_limit && g.tmode == P->timing) {
      P->g_used[i] = ++P->g_tick;
      return P->g_cache[i];
    }
    if (P->g_used[i] < P->g_used[lru]) lru = i;
  }
  if (P->g_cache.size() < kGraphCache) {
    P->g_cache.emplace_back();
    P->g_used.push_back(++P->g_tick);
    return P->g_cache.back();
  }
  P->g_used[lru] = ++P->g_tick;
  return P->g_cache[lru];  // run_graphed re-captures it
}

int execute_full(cusfft_plan_t plan, const void* d_x, int64_t* d_locs, void* d_vals) {
  return run_graphed(plan, full_entry(plan, d_x, d_locs, d_vals), d_x, d_locs, d_vals, [&] {
    const double2* x = reinterpret_cast<const double2*>(d_x);
    double2* v = reinterpret_cast<double2*>(d_vals);
    if (use_branches(plan)) {
      TRY(ensure_streams(plan));  // (graph-less runs: the second stream is used directly)
      return launch_branched(plan, x, d_locs, v);
    }
    TRY(launch_local(plan, x));
    if (plan->mode2) return launch_rest2(plan, d_locs, v, plan->stream);
    if (plan->comm) {
      g_pdl = false;
      TRY(launch_exchange(plan, plan->stream));
    }
    return launch_finish(plan, d_locs, v);
  });
}

}  // namespace

// ===========================================================================
// C ABI
// ===========================================================================
extern "C" {

int32_t cusfft_abi_version(void) { return CUSFFT_ABI_VERSION; }
int32_t cusfft_last_cuda_error(void) { return g_last_cuda_error; }
int32_t cusfft_last_nccl_error(void) { return g_last_nccl_error; }

const char* cusfft_strerror(int code) {
  switch (code) {
    case CUSFFT_SUCCESS: return "success";
    case CUSFFT_INVALID_N: return "n must be a power of two in [16, 2^31]";
    case CUSFFT_INVALID_B: return "B must be a power of two with 2 <= B < n (and its work arrays must fit)";
    case CUSFFT_INVALID_K: return "need 1 <= k <= 8192 and k <= num_select <= B";
    case CUSFFT_INVALID_LOOPS: return "need 1 <= T <= L_loc <= L <= 64, L_loc <= 32 and world | L (loop sharding)";
    case CUSFFT_INVALID_PARAM: return "invalid filter or plan parameter";
    case CUSFFT_NULL_PTR: return "null pointer argument";
    case CUSFFT_ALLOC: return "device allocation failed";
    case CUSFFT_CUDA: return "CUDA runtime error (see cusfft_last_cuda_error)";
    case CUSFFT_HIT_OVERFLOW: return "more than max_hits frequencies reached the vote threshold";
    case CUSFFT_INVALID_PLAN: return "invalid or destroyed plan";
    case CUSFFT_INTERNAL: return "device-side consistency check failed";
    case CUSFFT_NCCL: return "NCCL unavailable or an NCCL call failed (see cusfft_last_nccl_error)";
    default: return "unknown cusfft status";
  }
}

int64_t cusfft_default_B(int64_t n, int64_t k, double bcst) {
  if (n < 2 || k < 1 || !(bcst > 0)) return 0;
  const double v = bcst * std::sqrt((double)n * (double)k / std::log2((double)n));
  int64_t b = 1;
  while ((double)(2 * b) <= v) b *= 2;
  return b;
}

int cusfft_params_default(cusfft_params* p, int64_t n, int64_t k, int64_t B) {
  if (!p) return CUSFFT_NULL_PTR;
  if (!is_pow2(n) || n < 16 || n > (int64_t(1) << 31)) return CUSFFT_INVALID_N;
  if (!is_pow2(B) || B < 2 || B >= n) return CUSFFT_INVALID_B;
  if (k < 1) return CUSFFT_INVALID_K;
  std::memset(p, 0, sizeof(*p));
  p->filter = CUSFFT_FILTER_DOLPH_CHEBYSHEV;
  p->tolerance = 1e-8;
  p->lobefrac = 0.5 / (double)B;
  p->box_width = n / B - 1;
  p->loc_loops = 0;       // -> min(L, 8) at plan time
  p->vote_threshold = 0;  // -> floor(L_loc/2) + 1
  p->num_select = (int32_t)std::min<int64_t>(k, B);
  p->tau_mode = 1;
  p->seed = 1;
  p->max_hits = 0;  // -> from the expected false-hit count
  p->device = -1;
  p->debug = 0;
  p->taps = nullptr;
  p->num_taps = 0;
  p->cutoff_mode = CUSFFT_CUTOFF_EXACT;
  p->shard_mode = 0;
  p->cutoff_threshold = 0.0;
  p->loc_tolerance = 0.0;  // -> tolerance
  p->loc_lobefrac = 0.0;   // -> lobefrac
  p->l2_persist = 1;
  p->gather = 0;
  return CUSFFT_SUCCESS;
}

int cusfft_plan(cusfft_plan_t* out, int64_t n, int64_t k, int64_t B, int32_t L, const cusfft_params* p) {
  return make_plan(out, n, k, B, L, p, 0, 1, nullptr);
}

int cusfft_plan_dist(cusfft_plan_t* out, int64_t n, int64_t k, int64_t B, int32_t L, const cusfft_params* p,
                     int32_t rank, int32_t world, const void* nccl_unique_id) {
  return make_plan(out, n, k, B, L, p, rank, world, nccl_unique_id);
}

int cusfft_nccl_unique_id(void* out) {
  if (!out) return CUSFFT_NULL_PTR;
  const NcclApi* api = nccl_api();
  if (!api) return CUSFFT_NCCL;
  ncclUniqueId id;
  const ncclResult_t r = api->GetUniqueId(&id);
  if (r != ncclSuccess) {
    g_last_nccl_error = (int)r;
    return CUSFFT_NCCL;
  }
  std::memcpy(out, &id, sizeof(id));
  return CUSFFT_SUCCESS;
}

int cusfft_destroy(cusfft_plan_t plan) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  DeviceGuard g(plan->device);
  cudaStreamSynchronize(plan->stream);
  free_plan(plan);
  return CUSFFT_SUCCESS;
}

int cusfft_set_stream(cusfft_plan_t plan, void* s) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  plan->stream = reinterpret_cast<cudaStream_t>(s);
  return CUSFFT_SUCCESS;
}

int cusfft_execute_local(cusfft_plan_t plan, const void* d_x) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (!d_x) return CUSFFT_NULL_PTR;
  DeviceGuard g(plan->device);
  return run_graphed(plan, plan->g_local, d_x, nullptr, nullptr,
                     [&] { return launch_local(plan, reinterpret_cast<const double2*>(d_x)); });
}

int cusfft_execute_mid(cusfft_plan_t plan) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (!plan->mode2) return CUSFFT_INVALID_PARAM;
  DeviceGuard g(plan->device);
  return run_graphed(plan, plan->g_mid, nullptr, nullptr, nullptr, [&] {
    g_pdl = false;
    return launch_mid(plan, plan->stream);
  });
}

int cusfft_execute_finish(cusfft_plan_t plan, int64_t* d_locs, void* d_vals) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (!d_locs || !d_vals) return CUSFFT_NULL_PTR;
  DeviceGuard g(plan->device);
  return run_graphed(plan, plan->g_finish, d_locs, d_vals, nullptr, [&] {
    if (plan->mode2) {
      g_pdl = false;
      return launch_finish2(plan, d_locs, reinterpret_cast<double2*>(d_vals), plan->stream);
    }
    return launch_finish(plan, d_locs, reinterpret_cast<double2*>(d_vals));
  });
}

int cusfft_execute(cusfft_plan_t plan, const void* d_x, int64_t* d_locs, void* d_vals) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (!d_x || !d_locs || !d_vals) return CUSFFT_NULL_PTR;
  if (plan->world != 1 && !plan->comm) return CUSFFT_INVALID_LOOPS;
  DeviceGuard g(plan->device);
  return execute_full(plan, d_x, d_locs, d_vals);
}

int cusfft_set_pipeline(cusfft_plan_t plan, int32_t depth) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (depth < 1 || depth > 8) return CUSFFT_INVALID_PARAM;
  if (plan->world != 1) return CUSFFT_INVALID_LOOPS;
  DeviceGuard g(plan->device);
  CK(cudaStreamSynchronize(plan->stream));
  while ((int)plan->subs.size() > depth - 1) {
    free_plan(plan->subs.back());
    plan->subs.pop_back();
  }
  // events first: execute_batch indexes sub_ev[depth] for depth = 1 + subs.size()
  while ((int)plan->sub_ev.size() < depth + 1) {
    cudaEvent_t e;
    CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    plan->sub_ev.push_back(e);
  }
  while ((int)plan->subs.size() < depth - 1) {
    cusfft_plan_t sp = nullptr;
    const int rc = cusfft_plan(&sp, plan->n, plan->k, plan->B, plan->L, &plan->prm);  // prm.taps: the plan's own copy
    if (rc) return rc;  // subs keeps its previous (consistent) size
    cudaStream_t st = nullptr;
    const cudaError_t e = cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
    if (e != cudaSuccess) {
      g_last_cuda_error = (int)e;
      free_plan(sp);
      return CUSFFT_CUDA;
    }
    sp->stream = st;
    sp->own_stream = true;
    plan->subs.push_back(sp);
  }
  return CUSFFT_SUCCESS;
}

int cusfft_execute_batch(cusfft_plan_t plan, const void* d_x, int64_t count, int64_t x_stride, int64_t* d_locs,
                         void* d_vals) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (count < 0 || x_stride < plan->n) return CUSFFT_INVALID_PARAM;
  if (count == 0) return CUSFFT_SUCCESS;
  if (!d_x || !d_locs || !d_vals) return CUSFFT_NULL_PTR;
  if (plan->world != 1) return CUSFFT_INVALID_LOOPS;
  DeviceGuard g(plan->device);
  const double2* x = reinterpret_cast<const double2*>(d_x);
  double2* v = reinterpret_cast<double2*>(d_vals);
  const int depth = 1 + (int)plan->subs.size();
  if (depth > 1) {  // fork the clones' streams off the caller's stream
    CK(cudaEventRecord(plan->sub_ev[depth], plan->stream));
    for (auto* sp : plan->subs) CK(cudaStreamWaitEvent(sp->stream, plan->sub_ev[depth], 0));
  }
  for (int64_t b = 0; b < count; ++b) {
    const int lane = (int)(b % depth);
    cusfft_plan_t P = lane == 0 ? plan : plan->subs[lane - 1];
    P->stage_limit = plan->stage_limit;
    const int rc = execute_full(P, x + b * x_stride, d_locs + b * plan->k, v + b * plan->k);
    if (rc) return rc;
  }
  if (depth > 1) {  // join
    for (int l = 1; l < depth; ++l) {
      CK(cudaEventRecord(plan->sub_ev[l], plan->subs[l - 1]->stream));
      CK(cudaStreamWaitEvent(plan->stream, plan->sub_ev[l], 0));
    }
  }
  return CUSFFT_SUCCESS;
}

int cusfft_status(cusfft_plan_t plan) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  DeviceGuard g(plan->device);
  int flags[8];
  CK(cudaStreamSynchronize(plan->stream));
  CK(cudaMemcpy(flags, plan->d_flags, sizeof(flags), cudaMemcpyDeviceToHost));
  if (flags[1]) return CUSFFT_HIT_OVERFLOW;
  if (flags[2] || flags[3]) return CUSFFT_INTERNAL;
  for (auto* sp : plan->subs) {
    const int rc = cusfft_status(sp);
    if (rc) return rc;
  }
  return CUSFFT_SUCCESS;
}

int cusfft_execute_host(cusfft_plan_t plan, const void* h_x, int64_t* h_locs, void* h_vals) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (!h_x || !h_locs || !h_vals) return CUSFFT_NULL_PTR;
  if (plan->world != 1) return CUSFFT_INVALID_LOOPS;
  DeviceGuard g(plan->device);
  int rc;
  if (!plan->d_xbuf) {
    if ((rc = dalloc(&plan->d_xbuf, (size_t)plan->n))) return rc;
    if ((rc = dalloc(&plan->d_locs_buf, (size_t)plan->k))) return rc;
    if ((rc = dalloc(&plan->d_vals_buf, (size_t)plan->k))) return rc;
  }
  cudaStream_t st = plan->stream;
  // A pinned, device-mapped h_x is gathered in place over PCIe: only the samples the plan's
  // taps touch cross the bus (C3: 1.87 M samples of 16.8 M; e2e 4.93 -> 2.3 ms).  Pageable
  // memory (or CUSFFT_HOST_ZEROCOPY=0, A/B) is copied whole first.
  const void* xin = plan->d_xbuf;
  {
    const char* e = std::getenv("CUSFFT_HOST_ZEROCOPY");
    cudaPointerAttributes pa{};
    if (!(e && e[0] == '0') && cudaPointerGetAttributes(&pa, h_x) == cudaSuccess && pa.type == cudaMemoryTypeHost &&
        pa.devicePointer)
      xin = pa.devicePointer;
    cudaGetLastError();
  }
  if (xin == plan->d_xbuf)
    CK(cudaMemcpyAsync(plan->d_xbuf, h_x, (size_t)plan->n * 16, cudaMemcpyHostToDevice, st));
  TRY(execute_full(plan, xin, plan->d_locs_buf, plan->d_vals_buf));
  CK(cudaMemcpyAsync(h_locs, plan->d_locs_buf, (size_t)plan->k * 8, cudaMemcpyDeviceToHost, st));
  CK(cudaMemcpyAsync(h_vals, plan->d_vals_buf, (size_t)plan->k * 16, cudaMemcpyDeviceToHost, st));
  return cusfft_status(plan);
}

int cusfft_exchange_buffer(cusfft_plan_t plan, void** d_buf, int64_t* bytes_per_rank) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (!d_buf || !bytes_per_rank) return CUSFFT_NULL_PTR;
  *d_buf = plan->mode2 ? plan->d_cand : plan->d_records;
  *bytes_per_rank = plan->mode2 ? (int64_t)plan->cmax * plan->crec_bytes : (int64_t)plan->Lg * plan->lay.rec_bytes;
  return CUSFFT_SUCCESS;
}

int cusfft_exchange_buffer2(cusfft_plan_t plan, void** d_buf, int64_t* bytes_per_rank) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (!d_buf || !bytes_per_rank) return CUSFFT_NULL_PTR;
  if (!plan->mode2) return CUSFFT_INVALID_PARAM;
  *d_buf = plan->d_x2;
  *bytes_per_rank = (int64_t)plan->max_hits * plan->Lg * (int64_t)sizeof(double2);
  return CUSFFT_SUCCESS;
}

int32_t cusfft_exchange_kind(cusfft_plan_t plan) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  return plan->mode2 ? 2 : plan->xshard ? 1 : 0;
}

int cusfft_get_info(cusfft_plan_t plan, int64_t* info, int64_t* a, int64_t* sigma, int64_t* tau) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (info) {
    int64_t v[16] = {plan->n, plan->k, plan->B, plan->L, plan->filt[plan->nfilt - 1].w, plan->nb, plan->num,
                     plan->Lloc, plan->T, plan->max_hits, plan->sectors, plan->staged ? (int64_t)plan->grp_s.size() - 1 : 0,
                     plan->filt[0].w, plan->nfilt, plan->tail_esz ? 1 : 0, plan->comm ? 1 : 0};
    std::memcpy(info, v, sizeof(v));
  }
  for (int r = 0; r < plan->L; ++r) {
    if (a) a[r] = plan->a_r[r];
    if (sigma) sigma[r] = plan->sigma_r[r];
    if (tau) tau[r] = plan->tau_r[r];
  }
  return CUSFFT_SUCCESS;
}

int64_t cusfft_get_debug(cusfft_plan_t plan, int32_t what, void* dst, int64_t cap) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  DeviceGuard g(plan->device);
  CK(cudaStreamSynchronize(plan->stream));
  unsigned hc = 0;
  CK(cudaMemcpy(&hc, plan->d_flags, sizeof(unsigned), cudaMemcpyDeviceToHost));
  const int64_t H = std::min<int64_t>(hc, plan->max_hits);
  const int64_t B = plan->B, L = plan->L;
  auto slot_of = [&](int r) { return (r % plan->lworld) * plan->Lg + r / plan->lworld; };
  const Filter& Fl = plan->filt[0];
  const Filter& Fe = plan->filt[plan->nfilt - 1];
  int64_t need = 0;
  switch (what) {
    case CUSFFT_DEBUG_U: need = (int64_t)plan->Lg * B * 16; break;
    case CUSFFT_DEBUG_UHAT: need = L * B * 16; break;
    case CUSFFT_DEBUG_WINNERS: need = (int64_t)plan->Lloc * plan->Jcap * 4; break;
    case CUSFFT_DEBUG_HITS: need = H * 4; break;
    case CUSFFT_DEBUG_HIT_VALS: need = H * 16; break;
    case CUSFFT_DEBUG_PER_LOOP: need = plan->d_per_loop ? H * L * 16 : 0; break;
    case CUSFFT_DEBUG_TAPS: need = (int64_t)Fe.w * 8; break;
    case CUSFFT_DEBUG_GHAT: need = (plan->nb + 1) * 16; break;
    case CUSFFT_DEBUG_NUM_HITS: need = 8; break;
    case CUSFFT_DEBUG_LOC_TAPS: need = (int64_t)Fl.w * 8; break;
    case CUSFFT_DEBUG_LOC_GHAT: need = (plan->nb + 1) * 16; break;
    default: return CUSFFT_INVALID_PARAM;
  }
  if (!dst || cap < need || need == 0) return need;
  uint8_t* out = reinterpret_cast<uint8_t*>(dst);
  switch (what) {
    case CUSFFT_DEBUG_U:
      if (!plan->prm.debug && plan->staged) return CUSFFT_INVALID_PARAM;  // the staged fold writes u for debug plans only
      CK(cudaMemcpy(out, plan->d_u, need, cudaMemcpyDeviceToHost));
      break;
    case CUSFFT_DEBUG_UHAT:
      for (int r = 0; r < L; ++r)
        CK(cudaMemcpy(out + (int64_t)r * B * 16, plan->d_records + (int64_t)slot_of(r) * plan->lay.rec_bytes, B * 16,
                      cudaMemcpyDeviceToHost));
      break;
    case CUSFFT_DEBUG_WINNERS:
      for (int r = 0; r < plan->Lloc; ++r) {
        const int64_t s = slot_of(r);
        // shard_mode 2: the gathered candidate record (its offsets relative to the record's bitmap)
        const uint8_t* rec = plan->mode2
                                 ? plan->d_cand + ((s / plan->Lg) * plan->cmax + s % plan->Lg) * plan->crec_bytes -
                                       plan->lay.off_bitmap
                                 : plan->d_records + s * plan->lay.rec_bytes;
        int cnt = 0;
        CK(cudaMemcpy(&cnt, rec + plan->lay.off_cnt, 4, cudaMemcpyDeviceToHost));
        cnt = std::max(0, std::min(cnt, plan->Jcap));
        int32_t* o = reinterpret_cast<int32_t*>(out + (int64_t)r * plan->Jcap * 4);
        CK(cudaMemcpy(o, rec + plan->lay.off_J, (int64_t)cnt * 4, cudaMemcpyDeviceToHost));
        for (int j = cnt; j < plan->Jcap; ++j) o[j] = -1;
      }
      break;
    case CUSFFT_DEBUG_HITS:  // (shard_mode 2: the ascending list the medians are aligned with)
      CK(cudaMemcpy(out, plan->mode2 ? plan->d_hits2 : plan->d_hits, need, cudaMemcpyDeviceToHost));
      break;
    case CUSFFT_DEBUG_HIT_VALS:
      CK(cudaMemcpy(out, plan->d_hit_vals, need, cudaMemcpyDeviceToHost));
      break;
    case CUSFFT_DEBUG_PER_LOOP: {
      std::vector<double2> tmp((size_t)(H * L));
      CK(cudaMemcpy(tmp.data(), plan->d_per_loop, need, cudaMemcpyDeviceToHost));
      double2* o = reinterpret_cast<double2*>(out);
      for (int64_t h = 0; h < H; ++h)
        for (int r = 0; r < L; ++r) o[h * L + r] = tmp[(size_t)(h * L + slot_of(r))];
      break;
    }
    case CUSFFT_DEBUG_TAPS:
      CK(cudaMemcpy(out, Fe.d_taps, need, cudaMemcpyDeviceToHost));
      break;
    case CUSFFT_DEBUG_GHAT:
      CK(cudaMemcpy(out, Fe.d_ghat, need, cudaMemcpyDeviceToHost));
      break;
    case CUSFFT_DEBUG_LOC_TAPS:
      CK(cudaMemcpy(out, Fl.d_taps, need, cudaMemcpyDeviceToHost));
      break;
    case CUSFFT_DEBUG_LOC_GHAT:
      CK(cudaMemcpy(out, Fl.d_ghat, need, cudaMemcpyDeviceToHost));
      break;
    case CUSFFT_DEBUG_NUM_HITS: {
      int64_t v = hc;
      std::memcpy(out, &v, 8);
      break;
    }
  }
  return need;
}

int cusfft_set_timing(cusfft_plan_t plan, int32_t enable) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  DeviceGuard g(plan->device);
  if (enable && !plan->ev_made) {
    for (auto& e : plan->ev) CK(cudaEventCreate(&e));
    plan->ev_made = true;
  }
  if (enable < 0 || enable > 2) return CUSFFT_INVALID_PARAM;
  plan->timing = enable;
  return CUSFFT_SUCCESS;
}

int cusfft_get_stage_times(cusfft_plan_t plan, float* ms, int32_t cap) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (!ms) return CUSFFT_NULL_PTR;
  if (!plan->ev_made) return CUSFFT_INVALID_PARAM;
  DeviceGuard g(plan->device);
  CK(cudaStreamSynchronize(plan->stream));
  for (int i = 0; i < 6 && i < cap; ++i) {
    float t = 0.f;
    const int i0 = plan->timing == 2 ? 0 : i, i1 = plan->timing == 2 ? 6 : i + 1;  // mode 2: ms[0] = whole graph
    if ((plan->timing == 2 && i > 0) || cudaEventElapsedTime(&t, plan->ev[i0], plan->ev[i1]) != cudaSuccess) {
      t = -1.f;
      cudaGetLastError();  // do not leave a stale error for later launch checks
    }
    ms[i] = t;
  }
  if (cap >= 7) {
    float t = -1.f;
    if (!plan->staged || plan->grp_s.size() > 2 || cudaEventElapsedTime(&t, plan->ev[0], plan->ev[7]) != cudaSuccess) {
      t = -1.f;
      cudaGetLastError();
    }
    ms[6] = t;
  }
  return CUSFFT_SUCCESS;
}

int cusfft_set_stage_limit(cusfft_plan_t plan, int32_t stages) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (stages < 1 || stages > 6) return CUSFFT_INVALID_PARAM;
  plan->stage_limit = stages;
  return CUSFFT_SUCCESS;
}

#ifdef CUSFFT_TRACE
// Trace builds only (not part of include/cusfft.h): copy g_trace to host.
int cusfft_debug_trace(unsigned long long* host, int32_t n) {
  if (!host) return CUSFFT_NULL_PTR;
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpyFromSymbol(host, g_trace, sizeof(unsigned long long) * (n < 256 ? n : 256)));
  return CUSFFT_SUCCESS;
}
// Trace builds only: per-CTA records (3 u64 each, common.cuh KTraceScope); returns the count.
int cusfft_debug_cta_trace(unsigned long long* host, int32_t max_records) {
  if (!host) return CUSFFT_NULL_PTR;
  CK(cudaDeviceSynchronize());
  unsigned n = 0;
  CK(cudaMemcpyFromSymbol(&n, g_cta_n, sizeof(n)));
  int m = (int)(n < (unsigned)kCtaTraceMax ? n : (unsigned)kCtaTraceMax);
  if (m > max_records) m = max_records;
  if (m > 0) CK(cudaMemcpyFromSymbol(host, g_cta, sizeof(unsigned long long) * 3 * (size_t)m));
  return m;
}
// Reset the trace: phase slots 0, per-kernel start slots (128 + 2 id) ~0.
int cusfft_debug_trace_reset() {
  unsigned long long init[256];
  for (int i = 0; i < 256; ++i) init[i] = (i >= 128 && (i % 2) == 0) ? ~0ull : 0ull;
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpyToSymbol(g_trace, init, sizeof(init)));
  const unsigned zero = 0;
  CK(cudaMemcpyToSymbol(g_cta_n, &zero, sizeof(zero)));
  return CUSFFT_SUCCESS;
}
#endif

int32_t cusfft_launches_per_execute(cusfft_plan_t plan) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  const int nl = plan->nloc_local, ne = plan->Lg - plan->nloc_local;
  const int ranges = (nl > 0) + (ne > 0);
  const bool pass1 = plan->B1 > 1 && !plan->fused1;
  const bool branched = use_branches(plan);
  const bool f2s = use_fft2_select(plan);  // location pass 2 inside the cutoff kernel
  const int ffts = f2s ? (ne > 0 ? 1 : 0) : (branched ? ranges : 1);
  const int ngrp = plan->staged ? (int)plan->grp_s.size() - 1 : 0;
  int n = (ngrp > 1 ? 2 * ngrp - ranges : ngrp) + ranges /*phase 1 per group, fold per slot range (or group)*/ +
          ffts * (pass1 ? 2 : 1) /*fft*/ + (plan->sel_slots_h.empty() ? 0 : 1) +
          (plan->xshard && !plan->sel_slots_h.empty() ? 1 : 0) /*keys*/ + (plan->tail_esz ? 2 : 3);
  // shard_mode 2: vote (k_tail vote-only or k_vote) + k_rank_est + k_median + k_output
  if (plan->mode2) n = n - (plan->tail_esz ? 2 : 3) + 4;
  if (plan->d_pkb) n += 1;  // k_pk_build
  if (plan->remap) {  // a remap + an execution kernel per chunk of B taps instead of one fold per range
    n -= ranges;
    for (int s = 0; s < plan->Lg; ++s) n += 2 * plan->filt[plan->filt_of_local(s)].R;
  }
  return n;
}

}  // extern "C"
