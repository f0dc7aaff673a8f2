// cusfft.cu — plan construction, launch sequence and the C ABI declared in
// include/cusfft.h.  Host code runs only at plan time and to enqueue work;
// every step of the transform runs in the kernels of exec_kernels.cuh.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <utility>
#include <string>
#include <vector>

#include "../../include/cusfft.h"
#include "exec_kernels.cuh"
#include "plan_kernels.cuh"

using namespace cusfft;

namespace {

constexpr uint32_t kMagic = 0x5FF7B200u;
thread_local int g_last_cuda_error = 0;

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

}  // namespace

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
  int log2nb = 0, w = 0, R = 0, num = 0, Lloc = 0, T = 0, max_hits = 0;
  int Jcap = 0;  // winner-list capacity per loop (num, or B in THRESHOLD mode)
  int B1 = 1, B2 = 1, logB1 = 0, logB2 = 0;
  int kp2 = 1;
  int select_smem = 0, vote_smem = 0, output_smem = 0;
  int vote_grid = 1, est_grid = 1;
  int fft_smem1 = 0, fft_smem2 = 0;
  int fft_E = 512;                // elements per CTA of the FFT passes (CUSFFT_FFT_E=256|512|1024; 512 measured best at C3)
  std::vector<SlotParam> slots_h;       // slot order
  std::vector<int64_t> a_r, sigma_r, tau_r;  // loop order
  std::vector<int> loc_slots_h, sel_slots_h;
  RecLayout lay{};
  // device memory
  double* d_taps = nullptr;
  double* d_taps_perm = nullptr;  // fused fold+pass-1 layout (two-pass B, B1 <= 256)
  bool fused1 = false;
  // staged gather: address-sorted gather schedule of this rank
  bool staged = false;
  // Phase 2 variant (CUSFFT_STAGE_MODE): scatter = phase 1 writes each sample at
  // phase 2's position (coalesced phase 2) instead of in sorted order (read
  // through an index); split = phase 2 is a plain fold (k_fold_staged) followed
  // by the stand-alone FFT pass 1, instead of k_fold_fft1.
  bool stage_scatter = true;   // default: scatter staging + bulk-copy phase 2 (measured fastest)
  bool stage_split = false;
  bool stage_atomic = false;      // phase 1 multiplies by the tap and adds into u with fp64 L2 reductions, no staging
                                  // (CUSFFT_STAGE_MODE=atomic; bucket sums then not in Alg. 1's order: opt-in A/B)
  bool stage_packed = false;      // scatter schedule as packed (slot, i) words (k_stage_packed; CUSFFT_PACKED=0: off)
  int stage_ibits = 0;
  bool p2_tma = true;             // scatter phase 2 through bulk copies (k_fold_fft1_tma; CUSFFT_P2=ldg: k_fold_fft1 MODE 2)
  int stage_bs = 256;             // phase-1 CTA size (CUSFFT_STAGE_BS = 128: A/B)
  int stage_u = 4;                // gathers in flight per phase-1 thread (CUSFFT_STAGE_U = 2 / 4 / 8 / 16)
  bool p2_discard = false;        // CUSFFT_DISCARD=1: drop consumed staging lines from L2 (default keeps them:
                                  // the next execution's phase-1 stores then hit valid set-aside lines)
  bool slot_fused = false;        // FFT pass 2 (+ fold) + cutoff in one cluster kernel per slot (k_slot; CUSFFT_SLOT=1|2)
  bool slot_select = false;       // k_slot also runs the cutoff (cluster selection)
  bool slot_phase_a = false;      // k_slot also folds (phase A, CUSFFT_SLOT=2); default: after k_fold_fft1_tma
  int slot_smem = 0;
  int64_t sectors = 0;            // distinct 32-B sectors of x gathered by this rank (the fold's DRAM floor)
  // Slot groups, each with its own sorted schedule (default: one group of all
  // local slots; CUSFFT_STAGE_GROUPS=2 splits location / estimation loops,
  // which halves each staging buffer but costs phase-1 locality: slower on B200).
  struct StageGroup {
    int s0 = 0, s1 = 0;          // local slots [s0, s1)
    int64_t total = 0;           // (s1 - s0) * w samples
    uint32_t* spos = nullptr;    // [total] sorted gather positions
    uint32_t* inv = nullptr;     // [s1 - s0][R][B] staging index in the fused kernel's thread order (index mode)
    uint32_t* dst = nullptr;     // [total] thread-order staging position of sorted gather q (scatter mode)
    uint32_t* code = nullptr;    // [total] packed (local slot << ibits | i) in address order (packed scatter mode)
    double2* staging = nullptr;  // this group's staging buffer (groups share one unless branched)
  };
  std::vector<StageGroup> groups;
  double2* d_staging = nullptr;   // [max group total]
  cudaAccessPolicyWindow stage_window = {};
  bool setaside = false;          // holds a reference on the device's persisting-L2 set-aside  // persisting L2 window over d_staging
  double2* d_ghat = nullptr;
  double2* d_tw = nullptr;
  SlotParam* d_slots = nullptr;
  int* d_loc_slots = nullptr;
  uint32_t* d_loc_sigma = nullptr;
  uint32_t* d_loc_a = nullptr;
  int* d_sel_slots = nullptr;
  double2* d_u = nullptr;
  double2* d_v = nullptr;
  uint8_t* d_records = nullptr;
  uint64_t* d_keys = nullptr;     // [n_sel][B] cutoff keys of this rank's location loops
  uint32_t* d_hist = nullptr;     // [n_sel][4096] top-digit histograms (self-resetting)
  int* d_key_index = nullptr;     // [Lg] local slot -> selection index or -1
  uint32_t* d_ohist = nullptr;    // [4096] top-digit histogram of the output keys (self-resetting)
  uint32_t* d_hist1 = nullptr;    // [n_sel][4096] level-1 cutoff histograms (self-resetting)
  uint64_t* d_ckey = nullptr;     // [n_sel][kSelCap] cutoff boundary candidates
  int* d_cidx = nullptr;
  int* d_ccount = nullptr;        // [n_sel] candidate counters (self-resetting)
  int* d_done = nullptr;          // [n_sel] finished-CTA counters (self-resetting)
  int sel_S = 1;                  // CTAs per location loop in k_select
  bool pk_direct = false;         // the cutoff writes k_vote8's byte-per-bucket array (d_pk, in the zero block)
  uint32_t* d_pk = nullptr;
  bool vote_packed = false;       // k_vote8 (L_loc <= 8, B <= 16384; CUSFFT_VOTE_BITMAP=1 forces k_vote)
  int vote8_grid = 1;
  bool vote_pairs = true;         // k_vote8 pair enumeration when T > ceil(L_loc/2) (CUSFFT_VOTE_PAIRS=0: off)
  bool sel_multi = false;
  bool sel_cluster = false;       // k_select_cluster (256 <= B <= 65536; CUSFFT_SELECT=single|multi to A/B)         // force the multi-CTA k_select (CUSFFT_SELECT_MULTI=1); else k_select1 for B <= 65536
  int* d_hits = nullptr;
  double2* d_hit_vals = nullptr;
  uint64_t* d_hit_keys = nullptr;
  double2* d_per_loop = nullptr;
  int* d_zero = nullptr;   // per-execution block, zeroed by the first fold kernel of each execution:
  int nzero = 0;           //   flags[8] | hist0[n_sel][4096] | hist1[n_sel][4096] | ohist[4096] | ccount | done
  int* d_flags = nullptr;  // [0] hit_count (unsigned), [1] overflow, [2] select mismatch, [3] output mismatch
  double2* d_xbuf = nullptr;
  int64_t* d_locs_buf = nullptr;
  double2* d_vals_buf = nullptr;
  cudaStream_t stream = nullptr;
  bool own_stream = false;        // clone plans (batched execution) own their stream
  int device = 0;
  bool timing = false;
  cudaEvent_t ev[8] = {};  // stage boundaries 0..6; [7] after phase 1 of the staged fold
  bool ev_made = false;
  // CUDA graphs of the launch sequences, keyed by the caller's pointers
  bool use_graph = true;
  bool branched = false;          // two-branch graph (location chain || estimation folds); opt-in
  bool sel_local_pick = false;    // cluster cutoff picks the boundary bin per CTA (CUSFFT_SEL_LOCALPICK=1; slower)
  int est_p2_pad = 0;             // extra dynamic smem (bytes) of the estimation branch's phase 2 (CUSFFT_EST_P2_PAD)
  bool est_seg = true;            // k_estimate_seg for L <= 16 (CUSFFT_EST_SEG=0: k_estimate)
  bool code_ef = false;           // CUSFFT_CODE_EF=1: schedule words loaded evict_first (A/B)
  bool split_launch = false;      // CUSFFT_SPLIT_LAUNCH=1: phase 1 as a plain launch before the graph of the rest
  int branch_fork = 0;            // CUSFFT_BRANCH=2..5: the estimation branch forks after phase 1 / the location
                                  // slots' phase 2 / their FFT pass 2 / the cutoff
  bool branch_p2 = true;          // CUSFFT_BRANCH=2: one phase 1, then location chain || estimation phase 2 + FFT
  bool skip_stage = false;        // measurement only (CUSFFT_SKIP_STAGE)
  int stage_cps = 4;              // phase-1 CTAs per SM: one resident wave (occupancy query; CUSFFT_STAGE_CPS overrides)
  int nloc_local = 0;             // local slots [0, nloc_local) are location loops
  cudaStream_t cap_stream = nullptr, cap_stream2 = nullptr;
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  int stage_limit = 6;
  int cur_prio = 0, prio_hi = 0, prio_lo = 0;  // launch priorities (branched graph)
  struct GraphEntry {
    int lim = -1;
    const void* a = nullptr;
    const void* b = nullptr;
    const void* c = nullptr;
    cudaGraphExec_t exec = nullptr;
  } g_full, g_local, g_finish, g_full_t, g_local_t, g_finish_t;  // *_t: with timing event nodes
  // whole-transform graphs by (x, locs, vals): up to kGraphCache, least recently used replaced
  std::vector<GraphEntry> g_cache;
  std::vector<uint64_t> g_used;
  uint64_t g_tick = 0;
  // batched execution (cusfft_execute_batch): depth-1 clones of this plan, each on its own stream
  std::vector<cusfft_plan_s*> subs;
  std::vector<cudaEvent_t> sub_ev;  // [depth] join events (+ fork event at the end)
};

constexpr size_t kGraphCache = 64;

namespace {

bool valid_plan(cusfft_plan_t p) { return p && p->magic == kMagic; }

// B1 x B2 splits with a k_slot instantiation
bool slot_shape_ok(int B1, int B2) {
  return (B1 == 64 && (B2 == 32 || B2 == 64)) || (B1 == 128 && (B2 == 64 || B2 == 128)) ||
         (B1 == 256 && (B2 == 128 || B2 == 256));
}

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
// by the plans of a device: raised to the largest request while any plan holds
// it, restored to the value found before the first plan when the last one is
// destroyed, so other work on the device (e.g. dense cuFFT) gets the whole L2
// back.
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
  for (auto& g : p->groups) {
    if (g.spos) cudaFree(g.spos);
    if (g.inv) cudaFree(g.inv);
    if (g.dst) cudaFree(g.dst);
    if (g.code) cudaFree(g.code);
  }
  void* ptrs[] = {p->d_taps, p->d_taps_perm, p->d_staging, p->d_ghat, p->d_tw, p->d_slots, p->d_loc_slots, p->d_loc_sigma, p->d_loc_a,
                  p->d_sel_slots, p->d_u, p->d_v, p->d_records, p->d_keys, p->d_zero, p->d_key_index, p->d_ckey, p->d_cidx, p->d_hits, p->d_hit_vals,
                  p->d_hit_keys, p->d_per_loop, p->d_xbuf, p->d_locs_buf, p->d_vals_buf};
  for (void* q : ptrs)
    if (q) cudaFree(q);
  if (p->ev_made)
    for (auto& e : p->ev) cudaEventDestroy(e);
  for (auto* g : {&p->g_full, &p->g_local, &p->g_finish, &p->g_full_t, &p->g_local_t, &p->g_finish_t})
    if (g->exec) cudaGraphExecDestroy(g->exec);
  for (auto& g : p->g_cache)
    if (g.exec) cudaGraphExecDestroy(g.exec);
  for (auto* sp : p->subs) free_plan(sp);
  for (auto e : p->sub_ev) cudaEventDestroy(e);
  if (p->own_stream && p->stream) cudaStreamDestroy(p->stream);
  if (p->cap_stream) cudaStreamDestroy(p->cap_stream);
  if (p->cap_stream2) cudaStreamDestroy(p->cap_stream2);
  if (p->ev_fork) cudaEventDestroy(p->ev_fork);
  if (p->ev_join) cudaEventDestroy(p->ev_join);
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
  if (q.shard_mode != 0 && q.shard_mode != 1) return CUSFFT_INVALID_PARAM;
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
    if (q.box_width < 1 || q.box_width > n || (q.box_width % 2) == 0) return CUSFFT_INVALID_PARAM;
  }
  if (q.max_hits < 1 || q.max_hits > (int64_t(1) << 30)) return CUSFFT_INVALID_PARAM;
  if (q.cutoff_mode < CUSFFT_CUTOFF_EXACT || q.cutoff_mode > CUSFFT_CUTOFF_THRESHOLD) return CUSFFT_INVALID_PARAM;
  if (q.cutoff_mode == CUSFFT_CUTOFF_SORT && B > 16384) return CUSFFT_INVALID_PARAM;
  if (q.cutoff_mode == CUSFFT_CUTOFF_THRESHOLD && !(q.cutoff_threshold > 0.0)) return CUSFFT_INVALID_PARAM;
  if (q.tau_mode != 0 && q.tau_mode != 1) return CUSFFT_INVALID_PARAM;
  return CUSFFT_SUCCESS;
}

int64_t filter_len(const cusfft_params& q) {
  const double pi = 3.14159265358979323846;
  int64_t w;
  if (q.taps) return q.num_taps;
  if (q.filter == CUSFFT_FILTER_DOLPH_CHEBYSHEV)
    w = (int64_t)std::floor(std::acosh(1.0 / q.tolerance) / (pi * q.lobefrac));
  else
    w = (int64_t)std::floor(2.0 * std::log(1.0 / q.tolerance) / (pi * q.lobefrac));
  if (w % 2 == 0) --w;
  return w;
}

template <class T>
int dalloc(T** ptr, size_t count) {
  if (count == 0) count = 1;
  CK(cudaMalloc((void**)ptr, count * sizeof(T)));
  return CUSFFT_SUCCESS;
}

#define TRY(expr)              \
  do {                         \
    int rc_ = (expr);          \
    if (rc_ != CUSFFT_SUCCESS) \
      return rc_;              \
  } while (0)

int build_filter(cusfft_plan_t P) {
  const cusfft_params& q = P->prm;
  const int w = P->w;
  const int padded = P->R * (int)P->B;
  const int c = (w - 1) / 2;
  cudaStream_t st = P->stream;
  if (q.taps) {
    CK(cudaMemsetAsync(P->d_taps, 0, (size_t)padded * sizeof(double), st));
    CK(cudaMemcpyAsync(P->d_taps, q.taps, (size_t)w * sizeof(double), cudaMemcpyHostToDevice, st));
  } else {
    double* win = nullptr;
    double* pj = nullptr;
    TRY(dalloc(&win, (size_t)c + 1));
    if (q.filter == CUSFFT_FILTER_DOLPH_CHEBYSHEV) {
      TRY(dalloc(&pj, (size_t)c + 1));
      const double x0 = std::cosh(std::acosh(1.0 / q.tolerance) / (double)(w - 1));
      k_cheb_samples<<<(c + 256) / 256, 256, 0, st>>>(pj, w, x0);
      CKL();
      k_dc_window<<<c + 1, 256, 0, st>>>(pj, win, w);
      CKL();
    } else {
      const double s = (double)c / std::sqrt(2.0 * std::log(1.0 / q.tolerance));
      k_gauss_window<<<(c + 256) / 256, 256, 0, st>>>(win, w, s);
      CKL();
    }
    k_taps<<<(padded + 255) / 256, 256, 0, st>>>(win, P->d_taps, w, padded, P->n, q.box_width);
    CKL();
    k_normalize<<<1, 1024, 0, st>>>(P->d_taps, w);
    CKL();
    CK(cudaStreamSynchronize(st));
    cudaFree(win);
    if (pj) cudaFree(pj);
  }
  k_ghat<<<(int)P->nb + 1, 256, 0, st>>>(P->d_taps, P->d_ghat, w, P->n, (int)P->nb);
  CKL();
  k_twiddles<<<(int)((P->B + 255) / 256), 256, 0, st>>>(P->d_tw, (int)P->B);
  CKL();
  return CUSFFT_SUCCESS;
}

// Kernel launch carrying an explicit scheduling priority: stream priorities are
// not captured into graph kernel nodes, the launch attribute is.
// g_pdl: programmatic dependent launch for this launch (every hot kernel
// begins with pdl_wait(), so it may be launched while its predecessor drains).
thread_local bool g_pdl = false;
// g_apw: L2 access-policy window for this launch (persisting staging buffer).
thread_local cudaAccessPolicyWindow g_apw = {};

template <typename... KArgs, typename... Args>
cudaError_t launch_k(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, int prio,
                     Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[3];
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = prio;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = g_pdl ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  if (g_apw.num_bytes) {
    attr[2].id = cudaLaunchAttributeAccessPolicyWindow;
    attr[2].val.accessPolicyWindow = g_apw;
    cfg.numAttrs = 3;
  }
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// Elements per CTA of the batched B1/B2-point FFT passes: g_fft_E (1024
// default; CUSFFT_FFT_E=512|256 for more, smaller CTAs), at least M.
thread_local int g_fft_E = 1024;

template <int M, int E>
cudaError_t launch_fft_e(const FftPassArgs& a, int smem, cudaStream_t st, int prio) {
  constexpr int NSEQ = E / M;
  const int grid = (a.total_seq + NSEQ - 1) / NSEQ;
  return launch_k(k_fft<M, E, 128>, dim3(grid), dim3(128), fft_smem_bytes(E), st, prio, a);
}

template <int M>
cudaError_t launch_fft_t(const FftPassArgs& a, int smem, cudaStream_t st, int prio) {
  (void)smem;
  if constexpr (M >= 1024) {
    return launch_fft_e<M, M>(a, 0, st, prio);
  } else {
    if (g_fft_E <= 256 && M <= 256) return launch_fft_e<M, (M < 256 ? 256 : M)>(a, 0, st, prio);
    if (g_fft_E <= 512 && M <= 512) return launch_fft_e<M, 512>(a, 0, st, prio);
    return launch_fft_e<M, 1024>(a, 0, st, prio);
  }
}

cudaError_t launch_fft(int M, const FftPassArgs& a, int smem, cudaStream_t st, int prio = 0) {
  switch (M) {
    case 2: return launch_fft_t<2>(a, smem, st, prio);
    case 4: return launch_fft_t<4>(a, smem, st, prio);
    case 8: return launch_fft_t<8>(a, smem, st, prio);
    case 16: return launch_fft_t<16>(a, smem, st, prio);
    case 32: return launch_fft_t<32>(a, smem, st, prio);
    case 64: return launch_fft_t<64>(a, smem, st, prio);
    case 128: return launch_fft_t<128>(a, smem, st, prio);
    case 256: return launch_fft_t<256>(a, smem, st, prio);
    case 512: return launch_fft_t<512>(a, smem, st, prio);
    case 1024: return launch_fft_t<1024>(a, smem, st, prio);
    case 2048: return launch_fft_t<2048>(a, smem, st, prio);
    case 4096: return launch_fft_t<4096>(a, smem, st, prio);
    default: return cudaErrorInvalidValue;
  }
}

template <int M, int E>
cudaError_t set_fft_attr_e() {
  return cudaFuncSetAttribute(k_fft<M, E, 128>, cudaFuncAttributeMaxDynamicSharedMemorySize, fft_smem_bytes(E));
}

template <int M>
cudaError_t set_fft_attr_t() {
  if constexpr (M >= 1024) {
    return set_fft_attr_e<M, M>();
  } else {
    cudaError_t e = set_fft_attr_e<M, 1024>();
    if constexpr (M <= 512) {
      cudaError_t e2 = set_fft_attr_e<M, 512>();
      if (e2 != cudaSuccess) e = e2;
    }
    if constexpr (M <= 256) {
      cudaError_t e3 = set_fft_attr_e<M, (M < 256 ? 256 : M)>();
      if (e3 != cudaSuccess) e = e3;
    }
    return e;
  }
}

cudaError_t set_fft_attrs() {
  cudaError_t e = cudaSuccess;
  cudaError_t r[] = {set_fft_attr_t<2>(), set_fft_attr_t<4>(), set_fft_attr_t<8>(), set_fft_attr_t<16>(),
                     set_fft_attr_t<32>(), set_fft_attr_t<64>(), set_fft_attr_t<128>(), set_fft_attr_t<256>(),
                     set_fft_attr_t<512>(), set_fft_attr_t<1024>(), set_fft_attr_t<2048>(), set_fft_attr_t<4096>()};
  for (cudaError_t x : r)
    if (x != cudaSuccess) e = x;
  return e;
}

int make_plan(cusfft_plan_t* out, int64_t n, int64_t k, int64_t B, int32_t L, const cusfft_params* pin, int rank,
              int world) {
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
  {
    int rc = validate(n, k, B, L, q, rank, world);
    if (rc) return rc;
  }
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

  cusfft_plan_t P = new (std::nothrow) cusfft_plan_s();
  if (!P) return CUSFFT_ALLOC;
  P->n = n; P->k = k; P->B = B; P->L = L; P->prm = q; P->rank = rank; P->world = world;
  if (q.taps) {  // the caller keeps ownership of its array: keep a copy (cusfft_set_pipeline clones read it)
    P->user_taps.assign(q.taps, q.taps + q.num_taps);
    P->prm.taps = P->user_taps.data();
  }
  P->device = dev;
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
  const int64_t w64 = filter_len(q);
  if (w64 < 1 || w64 > (int64_t(1) << 30)) {
    free_plan(P);
    return CUSFFT_INVALID_PARAM;
  }
  P->w = (int)w64;
  P->R = (int)((w64 + B - 1) / B);
  P->stream = nullptr;
  if (const char* e = std::getenv("CUSFFT_NO_GRAPH")) P->use_graph = !(e[0] == '1');
  if (const char* e = std::getenv("CUSFFT_BRANCH")) {
    P->branched = (e[0] == '1');
    P->branch_p2 = (e[0] >= '2' && e[0] <= '5');  // 0: one serial chain, 1: the two-group staged graph
    if (P->branch_p2) P->branch_fork = e[0] - '2';
  }
  if (const char* e = std::getenv("CUSFFT_SELECT_MULTI")) P->sel_multi = (e[0] == '1');
  P->sel_cluster = B >= 256 && B <= 65536 && !P->sel_multi && q.cutoff_mode != CUSFFT_CUTOFF_SORT;
  if (const char* e = std::getenv("CUSFFT_SELECT")) {
    if (e[0] == 's') P->sel_cluster = false;                        // single CTA (k_select1)
    if (e[0] == 'm') { P->sel_cluster = false; P->sel_multi = true; }  // multi-CTA (k_select)
  }
  P->vote_packed = q.loc_loops <= 8 && B <= kPk && B >= 32;
  if (const char* e = std::getenv("CUSFFT_VOTE_BITMAP")) P->vote_packed = P->vote_packed && !(e[0] == '1');
  if (const char* e = std::getenv("CUSFFT_VOTE_PAIRS")) P->vote_pairs = !(e[0] == '0');
  // measurement only: skip the staged gather's phase 1 (valid only for a repeated x)
  if (const char* e = std::getenv("CUSFFT_SKIP_STAGE")) P->skip_stage = (e[0] == '1');
  {  // one resident wave of phase-1 CTAs (grid-stride loop), at most 4 per SM: with 4 gathers in flight per
     // thread that is 4096 per SM, measured best (C3: 81.5-81.9 us; 8 in flight at 4 per SM 83.6-83.9,
     // 4 in flight at 8 per SM 83.9-84.1, at 3 per SM 83.2-83.5, at 2 per SM 88.2-88.7)
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_stage_packed<4>, 256, 0) == cudaSuccess && occ > 0)
      P->stage_cps = std::min(occ, 4);
    cudaGetLastError();
  }
  if (P->branched) P->stage_cps = 2;
  if (const char* e = std::getenv("CUSFFT_STAGE_CPS")) P->stage_cps = std::max(1, std::atoi(e));
  if (const char* e = std::getenv("CUSFFT_STAGE_U")) P->stage_u = std::atoi(e);
  if (const char* e = std::getenv("CUSFFT_STAGE_BS")) P->stage_bs = std::atoi(e);
  if (const char* e = std::getenv("CUSFFT_P2")) P->p2_tma = std::string(e) != "ldg";
  if (const char* e = std::getenv("CUSFFT_DISCARD")) P->p2_discard = (e[0] == '1');
  {
    const char* e = std::getenv("CUSFFT_PDL_TRIGGER");
    // default: only the estimation lets the output CTA launch early (measured: -0.8 us at C3;
    // early-resident vote / estimate / FFT CTAs slow their predecessors)
    const int m = e ? std::atoi(e) : 32;
    cudaMemcpyToSymbol(c_pdl_trigger, &m, sizeof(int));
  }
  if (const char* e = std::getenv("CUSFFT_SEL_LOCALPICK")) P->sel_local_pick = (e[0] == '1');
  if (const char* e = std::getenv("CUSFFT_EST_P2_PAD")) P->est_p2_pad = std::max(0, std::atoi(e));
  if (const char* e = std::getenv("CUSFFT_EST_SEG")) P->est_seg = (e[0] != '0');
  if (const char* e = std::getenv("CUSFFT_CODE_EF")) P->code_ef = (e[0] == '1');
  if (const char* e = std::getenv("CUSFFT_SPLIT_LAUNCH")) P->split_launch = (e[0] == '1');
  if (const char* e = std::getenv("CUSFFT_FFT_E")) P->fft_E = std::max(256, std::min(1024, std::atoi(e)));

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
  std::vector<uint32_t> loc_sig, loc_a;
  for (int s = 0; s < L; ++s) {
    if ((int)P->slots_h[s].loop < P->Lloc) {
      P->loc_slots_h.push_back(s);
      loc_sig.push_back(P->slots_h[s].sigma);
      loc_a.push_back(P->slots_h[s].a);
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
  if (B <= 2048) {
    P->B1 = 1; P->B2 = (int)B;
  } else {
    const int lb = ilog2(B);
    P->B1 = 1 << ((lb + 1) / 2);
    P->B2 = (int)(B / P->B1);
  }
  P->logB1 = ilog2(P->B1);
  P->logB2 = ilog2(P->B2);
  P->select_smem = 4096 * 4 + 64 * 4 + kSelCap * 12;
  P->sel_S = (int)std::max<int64_t>(1, std::min<int64_t>(16, B / 2048));
  P->vote_smem = P->Lloc * (int)((B + 31) / 32) * 4;
  P->kp2 = 1;
  while (P->kp2 < k) P->kp2 <<= 1;
  P->output_smem = 4096 * 4 + 64 * 4 + kOutCap * 12 + 2 * P->kp2 * 8 + 2 * 1024 * 4;
  P->fft_smem1 = fft_smem_bytes(std::max(1024, P->B1));
  P->fft_smem2 = fft_smem_bytes(std::max(1024, P->B2));
  {
    const int64_t units = (int64_t)(P->Lloc - P->T + 1) * P->num;  // one warp per (q0, J) range
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    P->vote_grid = (int)std::max<int64_t>(1, std::min<int64_t>((units + 7) / 8, (int64_t)sms * 4));
    const int64_t units8 = (int64_t)std::max(P->Lloc - P->T + 1, P->Lloc / 2) * P->num;
    P->vote8_grid = (int)std::max<int64_t>(1, std::min<int64_t>((units8 + 31) / 32, (int64_t)sms));
    P->est_grid = std::max(1, std::min((P->max_hits + 7) / 8, sms * 4));
  }
  if (P->vote_smem > 200 * 1024) {
    free_plan(P);
    return CUSFFT_INVALID_B;
  }

  int rc = CUSFFT_SUCCESS;
  auto fail = [&](int code) {
    free_plan(P);
    return code;
  };
  if ((rc = dalloc(&P->d_taps, (size_t)P->R * B))) return fail(rc);
  if ((rc = dalloc(&P->d_ghat, (size_t)P->nb + 1))) return fail(rc);
  if ((rc = dalloc(&P->d_tw, (size_t)B))) return fail(rc);
  if ((rc = dalloc(&P->d_slots, (size_t)L))) return fail(rc);
  if ((rc = dalloc(&P->d_loc_slots, (size_t)P->Lloc))) return fail(rc);
  if ((rc = dalloc(&P->d_loc_sigma, (size_t)P->Lloc))) return fail(rc);
  if ((rc = dalloc(&P->d_loc_a, (size_t)P->Lloc))) return fail(rc);
  if ((rc = dalloc(&P->d_sel_slots, std::max<size_t>(1, P->sel_slots_h.size())))) return fail(rc);
  if ((rc = dalloc(&P->d_u, (size_t)P->Lg * B))) return fail(rc);
  if (P->B1 > 1 && (rc = dalloc(&P->d_v, (size_t)P->Lg * B))) return fail(rc);
  if ((rc = dalloc(&P->d_records, (size_t)L * P->lay.rec_bytes))) return fail(rc);
  {
    const size_t nsel = std::max<size_t>(1, P->sel_slots_h.size());
    if ((rc = dalloc(&P->d_keys, nsel * B))) return fail(rc);
    // per-execution counters and histograms: one block, zeroed by the first fold kernel
    // cutoff-built vote bytes: every location loop selected on this rank, cluster cutoff, k_vote8
    P->pk_direct = P->vote_packed && P->sel_cluster && P->sel_slots_h == P->loc_slots_h && B % 32 == 0 &&
                   !(std::getenv("CUSFFT_PK") && std::getenv("CUSFFT_PK")[0] == '0');
    const int pk_off = (8 + (int)(2 * nsel * 4096 + 4096 + 2 * nsel) + 3) & ~3;  // 16-B aligned (uint4 copies)
    P->nzero = P->pk_direct ? pk_off + (int)(B / 4) : 8 + (int)(2 * nsel * 4096 + 4096 + 2 * nsel);
    if ((rc = dalloc(&P->d_zero, (size_t)P->nzero))) return fail(rc);
    P->d_flags = P->d_zero;
    P->d_hist = reinterpret_cast<uint32_t*>(P->d_zero + 8);
    P->d_hist1 = P->d_hist + nsel * 4096;
    P->d_ohist = P->d_hist1 + nsel * 4096;
    P->d_ccount = reinterpret_cast<int*>(P->d_ohist + 4096);
    P->d_done = P->d_ccount + nsel;
    if (P->pk_direct) P->d_pk = reinterpret_cast<uint32_t*>(P->d_zero + pk_off);
    if ((rc = dalloc(&P->d_key_index, (size_t)P->Lg))) return fail(rc);

    if ((rc = dalloc(&P->d_ckey, nsel * kSelCap))) return fail(rc);
    if ((rc = dalloc(&P->d_cidx, nsel * kSelCap))) return fail(rc);

    std::vector<int> kidx(P->Lg, -1);
    for (size_t i = 0; i < P->sel_slots_h.size(); ++i) kidx[P->sel_slots_h[i] - lrank * P->Lg] = (int)i;
    if (cudaMemcpy(P->d_key_index, kidx.data(), P->Lg * sizeof(int), cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemset(P->d_zero, 0, (size_t)P->nzero * sizeof(int)) != cudaSuccess) {
      g_last_cuda_error = (int)cudaGetLastError();
      return fail(CUSFFT_CUDA);
    }
  }
  if ((rc = dalloc(&P->d_hits, (size_t)P->max_hits))) return fail(rc);
  if ((rc = dalloc(&P->d_hit_vals, (size_t)P->max_hits))) return fail(rc);
  if ((rc = dalloc(&P->d_hit_keys, (size_t)P->max_hits))) return fail(rc);
  if (q.debug && (rc = dalloc(&P->d_per_loop, (size_t)P->max_hits * L))) return fail(rc);
  auto upload = [&](void* dst, const void* src, size_t bytes) -> int {
    CK(cudaMemcpy(dst, src, bytes, cudaMemcpyHostToDevice));
    return CUSFFT_SUCCESS;
  };
  if ((rc = upload(P->d_slots, P->slots_h.data(), L * sizeof(SlotParam)))) return fail(rc);
  if ((rc = upload(P->d_loc_slots, P->loc_slots_h.data(), P->Lloc * sizeof(int)))) return fail(rc);
  if ((rc = upload(P->d_loc_sigma, loc_sig.data(), P->Lloc * sizeof(uint32_t)))) return fail(rc);
  if ((rc = upload(P->d_loc_a, loc_a.data(), P->Lloc * sizeof(uint32_t)))) return fail(rc);
  if (!P->sel_slots_h.empty() &&
      (rc = upload(P->d_sel_slots, P->sel_slots_h.data(), P->sel_slots_h.size() * sizeof(int))))
    return fail(rc);
  if (cudaMemset(P->d_records, 0, (size_t)L * P->lay.rec_bytes) != cudaSuccess ||
      false) {
    g_last_cuda_error = (int)cudaGetLastError();
    return fail(CUSFFT_CUDA);
  }
  // k_output needs up to 205 KB at k = 8192 (kp2 = 8192): allow the device's opt-in maximum
  int smem_optin = 200 * 1024;
  cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  if (set_fft_attrs() != cudaSuccess ||
      cudaFuncSetAttribute(k_select, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024) != cudaSuccess ||
      cudaFuncSetAttribute(k_select1, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024) != cudaSuccess ||
      cudaFuncSetAttribute(k_select_cluster, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024) != cudaSuccess ||
      cudaFuncSetAttribute(k_select_sort, cudaFuncAttributeMaxDynamicSharedMemorySize, 210 * 1024) != cudaSuccess ||
      cudaFuncSetAttribute(k_vote, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024) != cudaSuccess ||
      cudaFuncSetAttribute(k_output, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_optin) != cudaSuccess ||
      P->output_smem > smem_optin) {
    g_last_cuda_error = (int)cudaGetLastError();
    return fail(CUSFFT_CUDA);
  }
  if ((rc = build_filter(P))) return fail(rc);
  P->fused1 = P->B1 > 1 && P->B1 <= 256;
  if (P->fused1) {  // taps_perm[rr B + cta 256 + t] = g[j(cta, t) + rr B], j = c + B2 j1
    const int64_t padded = (int64_t)P->R * B;
    std::vector<double> g((size_t)padded), gp((size_t)padded);
    if (cudaMemcpy(g.data(), P->d_taps, padded * sizeof(double), cudaMemcpyDeviceToHost) != cudaSuccess) {
      g_last_cuda_error = (int)cudaGetLastError();
      return fail(CUSFFT_CUDA);
    }
    const int C = 256 / P->B1;
    for (int64_t rr = 0; rr < P->R; ++rr)
      for (int64_t cta = 0; cta < B / 256; ++cta)
        for (int t = 0; t < 256; ++t) {
          const int64_t cc = cta * C + t / P->B1, j1 = t % P->B1;
          gp[(size_t)(rr * B + cta * 256 + t)] = g[(size_t)(rr * B + cc + (int64_t)P->B2 * j1)];
        }
    if ((rc = dalloc(&P->d_taps_perm, (size_t)padded))) return fail(rc);
    if ((rc = upload(P->d_taps_perm, gp.data(), padded * sizeof(double)))) return fail(rc);
  }
  {  // distinct 32-B sectors (2 complex samples) of x this rank gathers
    std::vector<uint64_t> bits((size_t)((n / 2 + 63) / 64), 0ull);
    const uint32_t nm = (uint32_t)(n - 1);
    for (int sl = 0; sl < P->Lg; ++sl) {
      const SlotParam& sp = P->slots_h[(size_t)lrank * P->Lg + sl];
      for (int i = 0; i < P->w; ++i) {
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
  {
    const char* e = std::getenv("CUSFFT_NO_STAGE");
    const char* eg = std::getenv("CUSFFT_STAGE_GROUPS");
    std::vector<std::pair<int, int>> ranges;
    // two groups (location / estimation slots): opt-in, and always for the branched graph
    if (P->nloc_local > 0 && P->nloc_local < P->Lg && ((eg && eg[0] == '2') || P->branched))
      ranges = {{0, P->nloc_local}, {P->nloc_local, P->Lg}};
    else
      ranges = {{0, P->Lg}};
    if (const char* em = std::getenv("CUSFFT_STAGE_MODE")) {  // fused_index | fused_scatter | split_index | split_scatter
      const std::string m(em);
      P->stage_atomic = m == "atomic";
      P->stage_split = m.rfind("split", 0) == 0 || P->stage_atomic;
      P->stage_scatter = m.find("scatter") != std::string::npos || P->stage_atomic;
    }
    {  // packed (slot, i) schedule words: fused scatter mode when local slot and tap index fit 32 bits
      int ib = 1;
      while ((int64_t(1) << ib) < P->w) ++ib;
      int sb = 0;
      while ((1 << sb) < P->Lg) ++sb;
      const char* ep = std::getenv("CUSFFT_PACKED");
      P->stage_ibits = ib;
      P->stage_packed = P->stage_scatter && !P->stage_split && ib + sb <= 32 && !(ep && ep[0] == '0');
      if (P->stage_atomic && ib + sb > 32) P->stage_atomic = P->stage_split = false;
      P->stage_packed = P->stage_packed || P->stage_atomic;
    }
    int64_t maxtot = 0, sumtot = 0;  // staging elements: w per slot (index mode) or R B per slot (scatter mode)
    for (auto& r : ranges) {
      const int64_t t = (int64_t)(r.second - r.first) * (P->stage_scatter ? P->R * B : P->w);
      maxtot = std::max<int64_t>(maxtot, t);
      sumtot += t;
    }
    if (P->branched) maxtot = sumtot;  // concurrent groups: one staging buffer each
    // the staging buffer must be (mostly) L2-resident between the two phases
    // (the staging schedule gathers from the whole signal: not for signal-sharded plans)
    P->staged = P->fused1 && !P->xshard && maxtot * 16 <= (int64_t)64 << 20 && !(e && e[0] == '1');
    if (P->staged) {
      const uint32_t nm = (uint32_t)(n - 1);
      const int C = 256 / P->B1;
      for (auto& r : ranges) {
        cusfft_plan_s::StageGroup g;
        g.s0 = r.first;
        g.s1 = r.second;
        g.total = (int64_t)(g.s1 - g.s0) * P->w;
        std::vector<uint64_t> ev((size_t)g.total);
        for (int sl = g.s0; sl < g.s1; ++sl) {
          const SlotParam& sp = P->slots_h[(size_t)lrank * P->Lg + sl];
          for (int i = 0; i < P->w; ++i) {
            const uint32_t pos = (sp.sigma * (uint32_t)i + sp.tau) & nm;
            const uint64_t id = (uint64_t)(sl - g.s0) * P->w + i;
            ev[(size_t)id] = ((uint64_t)pos << 32) | id;
          }
        }
        std::sort(ev.begin(), ev.end());
        std::vector<uint32_t> spos((size_t)g.total), dst, inv, code;
        if (P->stage_packed)
          code.assign((size_t)g.total, 0u);
        else if (P->stage_scatter)
          dst.assign((size_t)g.total, 0u);
        else
          inv.assign((size_t)(g.s1 - g.s0) * P->R * B, 0u);
        for (int64_t q = 0; q < g.total; ++q) {
          spos[(size_t)q] = (uint32_t)(ev[(size_t)q] >> 32);
          const uint64_t id = ev[(size_t)q] & 0xFFFFFFFFull;
          const int64_t sl = (int64_t)(id / P->w), i = (int64_t)(id % P->w);
          const int64_t rr = i / B, j = i % B;
          const int64_t c = j % P->B2, j1 = j / P->B2;
          const int64_t cta = c / C, t = (c % C) * P->B1 + j1;
          const uint32_t tpos = (uint32_t)((sl * P->R + rr) * B + (P->stage_split ? j : cta * 256 + t));
          if (P->stage_packed)
            code[(size_t)q] = ((uint32_t)sl << P->stage_ibits) | (uint32_t)i;
          else if (P->stage_scatter)
            dst[(size_t)q] = tpos;
          else
            inv[(size_t)tpos] = (uint32_t)q;
        }
        P->groups.push_back(g);
        auto& gg = P->groups.back();
        if (P->stage_packed) {
          if ((rc = dalloc(&gg.code, code.size()))) return fail(rc);
          if ((rc = upload(gg.code, code.data(), code.size() * sizeof(uint32_t)))) return fail(rc);
        } else if ((rc = dalloc(&gg.spos, (size_t)g.total)) ||
                   (rc = upload(gg.spos, spos.data(), spos.size() * sizeof(uint32_t)))) {
          return fail(rc);
        }
        if (P->stage_packed) {
        } else if (P->stage_scatter) {
          if ((rc = dalloc(&gg.dst, dst.size()))) return fail(rc);
          if ((rc = upload(gg.dst, dst.data(), dst.size() * sizeof(uint32_t)))) return fail(rc);
        } else {
          if ((rc = dalloc(&gg.inv, inv.size()))) return fail(rc);
          if ((rc = upload(gg.inv, inv.data(), inv.size() * sizeof(uint32_t)))) return fail(rc);
        }
      }
      if ((rc = dalloc(&P->d_staging, P->stage_atomic ? (size_t)1 : (size_t)maxtot))) return fail(rc);
      {
        int64_t off = 0;
        for (auto& g : P->groups) {
          g.staging = P->d_staging + off;
          if (P->branched) off += (g.s1 - g.s0) * (P->stage_scatter ? (int64_t)P->R * B : (int64_t)P->w);
        }
      }
      // Persisting-L2 set-aside for the staging buffer (a device-wide limit: raised, never lowered).
      int maxp = 0;
      cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev);
      // The set-aside is what keeps the staging (stored evict_last = persisting) apart from the
      // evict_first stream of x: without it C3 takes 100 us instead of 87.
      // CUSFFT_APW=0 turns it off for that A/B.
      const bool apw = !(std::getenv("CUSFFT_APW") && std::getenv("CUSFFT_APW")[0] == '0');
      const size_t win = (P->stage_atomic || !apw) ? 0 : std::min<size_t>((size_t)maxtot * 16, (size_t)maxp);
      size_t want = win;  // CUSFFT_SETASIDE_MB: a larger set-aside than the staging buffer (A/B)
      if (const char* e = std::getenv("CUSFFT_SETASIDE_MB"))
        if (win > 0) want = std::min<size_t>((size_t)maxp, std::max<size_t>(win, (size_t)std::atoll(e) << 20));
      if (win > 0) setaside_acquire(dev, want);
      P->setaside = win > 0;
      P->stage_window.base_ptr = P->d_staging;
      // the access-policy window on the launches adds nothing measurable (CUSFFT_APW=1 to attach it)
      P->stage_window.num_bytes = (std::getenv("CUSFFT_APW") && std::getenv("CUSFFT_APW")[0] == '1') ? win : 0;
      P->stage_window.hitRatio = 1.0f;
      P->stage_window.hitProp = cudaAccessPropertyPersisting;
      P->stage_window.missProp = cudaAccessPropertyStreaming;
    }
  }
  {  // fused slot kernel (k_slot): scatter-staged plans whose B1 x B2 split has an instantiation
    const char* e = std::getenv("CUSFFT_SLOT");
    const bool shape = slot_shape_ok(P->B1, P->B2);
    P->slot_smem = shape ? slot_smem_bytes(P->B1, P->B2, P->R) : 0;
    // opt-in (CUSFFT_SLOT=1: FFT pass 2 + cutoff fused; 2: also the fold): measured no faster
    // than the separate kernels on B200, kept for the A/B
    P->slot_phase_a = e && e[0] == '2';
    P->slot_fused = P->staged && P->stage_scatter && !P->stage_split && shape &&
                    (!P->slot_phase_a || P->slot_smem <= 220 * 1024) && e && (e[0] == '1' || e[0] == '2');
    P->slot_select = P->slot_fused && P->sel_cluster && !P->sel_slots_h.empty();
  }
  if (cudaStreamSynchronize(P->stream) != cudaSuccess) {
    g_last_cuda_error = (int)cudaGetLastError();
    return fail(CUSFFT_CUDA);
  }
  *out = P;
  return CUSFFT_SUCCESS;
}

template <int B1T, int B2T, bool FV>
cudaError_t launch_slot_t(cusfft_plan_t P, const SlotArgs& a, int nslots, cudaStream_t st) {
  static thread_local bool attr_set = false;
  if (!attr_set) {
    cudaFuncSetAttribute(k_slot<B1T, B2T, FV>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    attr_set = true;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(nslots * kSlotCS));
  cfg.blockDim = dim3(256);
  cfg.dynamicSmemBytes = FV ? (size_t)slot_smem_bytes_v(B1T, B2T) : (size_t)P->slot_smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[3];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = kSlotCS;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = g_pdl ? 1 : 0;
  attr[2].id = cudaLaunchAttributePriority;
  attr[2].val.priority = P->cur_prio;
  cfg.attrs = attr;
  cfg.numAttrs = 3;
  return cudaLaunchKernelEx(&cfg, k_slot<B1T, B2T, FV>, a);
}

// extra dynamic smem of the next bulk-copy phase-2 launch (fewer CTAs per SM)
thread_local int g_p2_pad = 0;

template <int B1T>
cudaError_t launch_fold_fft1_t(cusfft_plan_t P, const double2* x, const uint32_t* inv, const SlotParam* sp, double2* u,
                               double2* v, int nslots, ZeroArgs z, cudaStream_t st, bool staged_tord) {
  dim3 grid((unsigned)(P->B / 256), (unsigned)nslots);
  if (inv)  // staged: x is the staging buffer of the group, inv its index
    return launch_k(k_fold_fft1<B1T, 16, 1>, grid, dim3(256), 0, st, P->cur_prio, x, inv,
                    (const double*)P->d_taps_perm, sp, u, v, (const double2*)P->d_tw,
                    (int)P->B, P->B2, P->w, P->R, (uint32_t)(P->n - 1), 0u, (uint32_t)P->n, z);
  if (staged_tord && P->p2_tma && P->R <= 48) {  // staged in thread order, rows moved by bulk copies
    const size_t smem = (size_t)P->R * 4096 + (size_t)g_p2_pad;
    static thread_local bool attr_set = false;  // one flag per B1T instantiation
    if (!attr_set) {  // static + dynamic smem may exceed the 48 KB default
      cudaFuncSetAttribute(k_fold_fft1_tma<B1T>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
      attr_set = true;
    }
    return launch_k(k_fold_fft1_tma<B1T>, grid, dim3(256), smem, st, P->cur_prio, x,
                    (const double*)P->d_taps_perm, P->prm.debug ? u : nullptr, v, (const double2*)P->d_tw, (int)P->B, P->B2, P->w, P->R,
                    (int)P->p2_discard, z);
  }
  if (staged_tord)  // staged in thread order: x is the group's staging buffer
    return launch_k(k_fold_fft1<B1T, 16, 2>, grid, dim3(256), 0, st, P->cur_prio, x, (const uint32_t*)nullptr,
                    (const double*)P->d_taps_perm, sp, u, v, (const double2*)P->d_tw,
                    (int)P->B, P->B2, P->w, P->R, (uint32_t)(P->n - 1), 0u, (uint32_t)P->n, z);
  return launch_k(k_fold_fft1<B1T, 8, 0>, grid, dim3(256), 0, st, P->cur_prio, x, (const uint32_t*)nullptr,
                  (const double*)P->d_taps_perm, sp, u, v, (const double2*)P->d_tw, (int)P->B, P->B2, P->w, P->R,
                  (uint32_t)(P->n - 1), P->xlo, P->xspan, z);
}

cudaError_t launch_fold_fft1(cusfft_plan_t P, const double2* x, const uint32_t* inv, const SlotParam* sp, double2* u,
                             double2* v, int nslots, ZeroArgs z, cudaStream_t st, bool staged_tord = false) {
  switch (P->B1) {
    case 64: return launch_fold_fft1_t<64>(P, x, inv, sp, u, v, nslots, z, st, staged_tord);
    case 128: return launch_fold_fft1_t<128>(P, x, inv, sp, u, v, nslots, z, st, staged_tord);
    case 256: return launch_fold_fft1_t<256>(P, x, inv, sp, u, v, nslots, z, st, staged_tord);
    default: return cudaErrorInvalidValue;
  }
}

// The bulk-copy fold + FFT pass 1 writes u only for debug plans (the FFT reads v).
inline bool u_debug_only(cusfft_plan_t P) {
  return P->staged && P->stage_scatter && !P->stage_split && P->p2_tma && P->R <= 48 && !(P->slot_fused && P->slot_phase_a);
}

inline void mark(cusfft_plan_t P, int i) {
  if (P->timing) cudaEventRecord(P->ev[i], P->stream);
}

// Staged fold, phase 1: address-sorted gather of the group's samples into its staging buffer.
int launch_stage1(cusfft_plan_t P, const cusfft_plan_s::StageGroup& g, const double2* x, cudaStream_t st, ZeroArgs z) {
  if (P->skip_stage) return CUSFFT_SUCCESS;
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, P->device);
  const int tot = (int)g.total;
  const int per = 256 * std::max(1, P->stage_u);
  const int grid = std::max(1, std::min((tot + per - 1) / per, sms * P->stage_cps));
  g_apw = P->stage_window;  // keep the staging buffer L2-resident for phase 2
  cudaError_t e;
  if (g.code && P->stage_atomic) {
    double2* u = P->d_u + (size_t)g.s0 * P->B;
    CK(cudaMemsetAsync(u, 0, (size_t)(g.s1 - g.s0) * P->B * sizeof(double2), st));
    StagePackArgs a{x, g.code, nullptr, P->d_slots + (size_t)P->lrank * P->Lg + g.s0, tot, g.s1 - g.s0,
                    P->stage_ibits, P->R, ilog2(P->B), P->logB2, P->logB1, ilog2(256 / P->B1),
                    (uint32_t)(P->n - 1), z};
    e = launch_k(k_stage_atomic, dim3(grid), dim3(256), 0, st, P->cur_prio, a, (const double*)P->d_taps, u);
  } else if (g.code) {
    StagePackArgs a{x, g.code, g.staging, P->d_slots + (size_t)P->lrank * P->Lg + g.s0, tot, g.s1 - g.s0,
                    P->stage_ibits, P->R, ilog2(P->B), P->logB2, P->logB1, ilog2(256 / P->B1),
                    (uint32_t)(P->n - 1), z, P->code_ef ? 1 : 0};
    // CUSFFT_STAGE_BS = 128: half-size CTAs (A/B; the grid keeps the same threads per SM)
    const int bs = P->stage_bs == 128 ? 128 : 256;
    const dim3 gr((unsigned)(bs == 128 ? 2 * grid : grid)), bl((unsigned)bs);
    if (P->stage_u == 2)
      e = launch_k(k_stage_packed<2>, gr, bl, 0, st, P->cur_prio, a);
    else if (P->stage_u == 16)
      e = launch_k(k_stage_packed<16>, gr, bl, 0, st, P->cur_prio, a);
    else if (P->stage_u == 8)
      e = launch_k(k_stage_packed<8>, gr, bl, 0, st, P->cur_prio, a);
    else
      e = launch_k(k_stage_packed<4>, gr, bl, 0, st, P->cur_prio, a);
  } else {
    e = launch_k(k_stage, dim3(grid), dim3(256), 0, st, P->cur_prio, x, (const uint32_t*)g.spos,
                 (const uint32_t*)g.dst, g.staging, tot, z);
  }
  g_apw = cudaAccessPolicyWindow{};
  CK(e);
  return CUSFFT_SUCCESS;
}

// Staged fold, phase 2: the fold (+ FFT pass 1) of the group's slots from its staging buffer.
int launch_stage2(cusfft_plan_t P, const cusfft_plan_s::StageGroup& g, cudaStream_t st, ZeroArgs z) {
  const int B = (int)P->B;
  g_pdl = !P->timing;
  cudaError_t e;
  if (P->stage_atomic) return CUSFFT_SUCCESS;  // phase 1 already summed the buckets into u
  if (P->stage_split) {
    dim3 grid2((unsigned)(B / 256), (unsigned)(g.s1 - g.s0));
    if (g.dst)
      e = launch_k(k_fold_staged<true>, grid2, dim3(256), 0, st, P->cur_prio, (const double2*)g.staging,
                   (const uint32_t*)nullptr, (const double*)P->d_taps, P->d_u + (size_t)g.s0 * B, B, P->w, P->R, z);
    else
      e = launch_k(k_fold_staged<false>, grid2, dim3(256), 0, st, P->cur_prio, (const double2*)g.staging,
                   (const uint32_t*)g.inv, (const double*)P->d_taps, P->d_u + (size_t)g.s0 * B, B, P->w, P->R, z);
  } else {
    e = launch_fold_fft1(P, g.staging, g.inv, P->d_slots + (size_t)P->lrank * P->Lg + g.s0,
                         P->d_u + (size_t)g.s0 * B, P->d_v + (size_t)g.s0 * B, g.s1 - g.s0, z, st, g.dst != nullptr || g.code != nullptr);
  }
  CK(e);
  return CUSFFT_SUCCESS;
}

SelArgs make_sel_args(cusfft_plan_t P);

// Steps 2-4 of a staged group in the fused cluster kernel (do_select: with the cutoff).
int launch_slot(cusfft_plan_t P, const cusfft_plan_s::StageGroup& g, cudaStream_t st, bool do_select) {
  const int B = (int)P->B;
  SlotArgs a{};
  a.staging = g.staging;
  a.taps_perm = P->d_taps_perm;
  a.u = P->d_u + (size_t)g.s0 * B;
  a.recs = P->d_records + ((int64_t)P->lrank * P->Lg + g.s0) * P->lay.rec_bytes;
  a.rec_bytes = P->lay.rec_bytes;
  a.tw = P->d_tw;
  a.key_index = P->sel_slots_h.empty() ? nullptr : P->d_key_index + g.s0;
  a.keys = P->d_keys;
  a.hist = P->d_hist;
  a.B = B;
  a.w = P->w;
  a.R = P->R;
  a.discard = P->p2_discard ? 1 : 0;
  a.do_select = do_select ? 1 : 0;
  a.sel = make_sel_args(P);
  g_pdl = !P->timing;
  const int ns = g.s1 - g.s0;
  cudaError_t e = cudaErrorInvalidValue;
  const bool fv = !P->slot_phase_a;
  a.v = P->d_v + (size_t)g.s0 * B;
  switch (P->B1 * 1000 + P->B2) {
#define SLOT_CASE(b1, b2) \
  case b1 * 1000 + b2: e = fv ? launch_slot_t<b1, b2, true>(P, a, ns, st) : launch_slot_t<b1, b2, false>(P, a, ns, st); break;
    SLOT_CASE(64, 32)
    SLOT_CASE(64, 64)
    SLOT_CASE(128, 64)
    SLOT_CASE(128, 128)
    SLOT_CASE(256, 128)
    SLOT_CASE(256, 256)
#undef SLOT_CASE
    default: break;
  }
  CK(e);
  return CUSFFT_SUCCESS;
}

// Steps 1+2 (and the fused FFT pass 1) for this rank's local slots [s0, s1).
// zero_block: this launch also zeroes the per-execution block (first fold only).
int launch_fold(cusfft_plan_t P, const double2* x, int s0, int s1, cudaStream_t st, bool zero_block) {
  if (s1 <= s0) return CUSFFT_SUCCESS;
  const int B = (int)P->B;
  const SlotParam* sp = P->d_slots + (size_t)P->lrank * P->Lg + s0;
  ZeroArgs z{zero_block ? P->d_zero : nullptr, zero_block ? P->nzero : 0};
  if (P->staged) {  // per slot group: phase 1 (address-sorted gather into staging), phase 2 (fused fold)
    for (const auto& g : P->groups) {
      if (g.s1 <= s0 || g.s0 >= s1) continue;  // callers pass whole groups
      int rc;
      if ((rc = launch_stage1(P, g, x, st, z))) return rc;
      if (&g == &P->groups.front()) mark(P, 7);
      if (!P->skip_stage) z = ZeroArgs{nullptr, 0};
      if ((rc = launch_stage2(P, g, st, z))) return rc;
    }
  } else if (P->fused1) {
    CK(launch_fold_fft1(P, x, nullptr, sp, P->d_u + (size_t)s0 * B, P->d_v + (size_t)s0 * B, s1 - s0, z, st));
  } else {
    dim3 grid((B + 255) / 256, s1 - s0);
    CK(launch_k(k_fold<16>, grid, dim3(256), 0, st, P->cur_prio, x, (const double*)P->d_taps, sp,
                P->d_u + (size_t)s0 * B, B, P->w, P->R, (uint32_t)(P->n - 1), P->xlo, P->xspan, z));
  }
  return CUSFFT_SUCCESS;
}

// Step 3 (remaining FFT passes, cutoff keys) for local slots [s0, s1).
int launch_bfft(cusfft_plan_t P, int s0, int s1, cudaStream_t st) {
  if (s1 <= s0) return CUSFFT_SUCCESS;
  const int B = (int)P->B;
  const int ns = s1 - s0;
  g_fft_E = P->fft_E;
  double2* rec = reinterpret_cast<double2*>(P->d_records + ((int64_t)P->lrank * P->Lg + s0) * P->lay.rec_bytes);
  const int64_t rec_e = P->lay.rec_bytes / 16;
  // signal-sharded: the spectra are partial here, keys come after the all-reduce (launch_keys)
  const int* kidx = (P->sel_slots_h.empty() || P->xshard) ? nullptr : P->d_key_index + s0;
  if (P->B1 > 1) {
    if (!P->fused1 || (P->staged && P->stage_split)) {  // pass 1: B1-point FFTs over columns c (stride B2), twiddle e^{-2 pi i c k1 / B}
      FftPassArgs a1{P->d_u + (size_t)s0 * B, P->d_v + (size_t)s0 * B, P->d_tw, B, P->logB2, ns * P->B2, B, B, 1,
                     P->B2, 1, P->B2, 1, nullptr, nullptr, nullptr};
      CK(launch_fft(P->B1, a1, P->fft_smem1, st, P->cur_prio));
    }
    // pass 2: B2-point FFTs of contiguous rows k1, out to u^[k1 + B1 k2] (+ cutoff keys)
    FftPassArgs a2{P->d_v + (size_t)s0 * B, rec, P->d_tw, B, P->logB1, ns * P->B1, B, rec_e, P->B2, 1, 1, P->B1, 0,
                   kidx, P->d_keys, P->d_hist};
    CK(launch_fft(P->B2, a2, P->fft_smem2, st, P->cur_prio));
  } else {
    FftPassArgs a{P->d_u + (size_t)s0 * B, rec, P->d_tw, B, 0, ns, B, rec_e, 0, 1, 0, 1, 0, kidx, P->d_keys,
                  P->d_hist};
    CK(launch_fft(P->B2, a, P->fft_smem2, st, P->cur_prio));
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
  sa.S = P->sel_S;
  sa.keys = P->d_keys;
  sa.hist0 = P->d_hist;
  sa.hist1 = P->d_hist1;
  sa.ckey = P->d_ckey;
  sa.cidx = P->d_cidx;
  sa.ccount = P->d_ccount;
  sa.done = P->d_done;
  sa.status = P->d_flags + 1;
  sa.pk = P->d_pk;
  sa.local_pick = P->sel_local_pick ? 1 : 0;
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
  if (P->prm.cutoff_mode == CUSFFT_CUTOFF_SORT) {
    const int smem = (int)P->B * 12 + (int)((P->B + 31) / 32) * 4;
    CK(launch_k(k_select_sort, dim3((int)P->sel_slots_h.size()), dim3(1024), smem, st, P->cur_prio, sa));
    return CUSFFT_SUCCESS;
  }
  if (P->sel_cluster) {
    const int smem = (int)sizeof(SelClusterSmem) + (int)(P->B / kSelCL / 32) * 4;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(P->sel_slots_h.size() * kSelCL));
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
  if (P->B <= kSel1MaxB && !P->sel_multi) {
    const int smem = 4096 * 4 + 64 * 4 + kSelCap * 12 + (int)((P->B + 31) / 32) * 4;
    CK(launch_k(k_select1, dim3((int)P->sel_slots_h.size()), dim3(1024), smem, st, P->cur_prio, sa));
    return CUSFFT_SUCCESS;
  }
  CK(launch_k(k_select, dim3((int)P->sel_slots_h.size() * P->sel_S), dim3(kSelNT), P->select_smem, st, P->cur_prio,
              sa));
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

int launch_local(cusfft_plan_t P, const double2* x) {
  cudaStream_t st = P->stream;
  int rc;
  mark(P, 0);
  g_pdl = false;  // the first kernel follows arbitrary caller work
  if (P->slot_fused) {  // phase 1 per group, then one cluster kernel per group for steps 2-4
    ZeroArgs z{P->d_zero, P->nzero};
    for (const auto& g : P->groups) {  // stage 1 "fold": phase 1 (+ phase 2 unless k_slot folds)
      if ((rc = launch_stage1(P, g, x, st, z))) return rc;
      z = ZeroArgs{nullptr, 0};
      g_pdl = !P->timing;
      if (!P->slot_phase_a && (rc = launch_stage2(P, g, st, z))) return rc;
    }
    mark(P, 1);
    if (P->stage_limit < 2) return CUSFFT_SUCCESS;
    const bool sel = P->slot_select && P->stage_limit >= 3 && !P->xshard;
    for (const auto& g : P->groups)
      if ((rc = launch_slot(P, g, st, sel))) return rc;
    mark(P, 2);
    if (P->stage_limit < 3 || P->xshard) return CUSFFT_SUCCESS;
    if (!sel && (rc = launch_select(P, st))) return rc;
    mark(P, 3);
    return CUSFFT_SUCCESS;
  }
  rc = launch_fold(P, x, 0, P->Lg, st, true);
  g_pdl = !P->timing;
  if (rc) return rc;
  mark(P, 1);
  if (P->stage_limit < 2) return CUSFFT_SUCCESS;
  if ((rc = launch_bfft(P, 0, P->Lg, st))) return rc;
  mark(P, 2);
  if (P->stage_limit < 3 || P->xshard) return CUSFFT_SUCCESS;  // signal-sharded: cutoff after the all-reduce
  if ((rc = launch_select(P, st))) return rc;
  mark(P, 3);
  return CUSFFT_SUCCESS;
}

int launch_vote(cusfft_plan_t P, cudaStream_t st) {
  VoteArgs va;
  for (int q = 0; q < P->Lloc; ++q) {
    const uint8_t* rec = P->d_records + (int64_t)P->loc_slots_h[q] * P->lay.rec_bytes;
    va.bmp[q] = reinterpret_cast<const uint32_t*>(rec + P->lay.off_bitmap);
    va.Jp[q] = reinterpret_cast<const int*>(rec + P->lay.off_J);
    va.cntp[q] = reinterpret_cast<const int*>(rec + P->lay.off_cnt);
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
  va.pairs = (P->vote_pairs && P->T > (P->Lloc + 1) / 2) ? 1 : 0;
  va.hits = P->d_hits;
  va.hit_count = reinterpret_cast<unsigned*>(P->d_flags);
  va.max_hits = P->max_hits;
  va.pk = P->d_pk;
  if (P->vote_packed) {  // L_loc <= 8, B <= kPk: byte-per-bucket probes, one CTA per SM
    CK(launch_k(k_vote8, dim3(P->vote8_grid), dim3(1024), 0, st, P->cur_prio, va));
    return CUSFFT_SUCCESS;
  }
  CK(launch_k(k_vote, dim3(P->vote_grid), dim3(256), P->vote_smem, st, P->cur_prio, va));
  return CUSFFT_SUCCESS;
}

int launch_estimate(cusfft_plan_t P, cudaStream_t st) {
  EstArgs ea;
  ea.records = P->d_records;
  ea.lay = P->lay;
  ea.slots = P->d_slots;
  ea.L = P->L;
  ea.ghat = P->d_ghat;
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
  // segmented kernel (2 hits per warp at L = 16, 4 at L <= 8); CUSFFT_EST_SEG=0: warp per hit
  if (P->est_seg && P->L <= 8) {
    CK(launch_k(k_estimate_seg<8>, dim3(P->est_grid), dim3(256), 0, st, P->cur_prio, ea));
  } else if (P->est_seg && P->L <= 16) {
    CK(launch_k(k_estimate_seg<16>, dim3(P->est_grid), dim3(256), 0, st, P->cur_prio, ea));
  } else {
    CK(launch_k(k_estimate, dim3(P->est_grid), dim3(256), 0, st, P->cur_prio, ea));
  }
  return CUSFFT_SUCCESS;
}

int launch_output(cusfft_plan_t P, int64_t* locs, double2* vals, cudaStream_t st) {
  CK(launch_k(k_output, dim3(1), dim3(1024), P->output_smem, st, P->cur_prio, (const int*)P->d_hits,
              reinterpret_cast<const unsigned*>(P->d_flags), P->max_hits, (const double2*)P->d_hit_vals,
              (const uint64_t*)P->d_hit_keys, P->d_ohist, (int)P->k, P->kp2, ilog2(P->n), locs, vals,
              P->d_flags + 1));
  return CUSFFT_SUCCESS;
}

int launch_finish(cusfft_plan_t P, int64_t* locs, double2* vals) {
  cudaStream_t st = P->stream;
  int rc;
  g_pdl = !P->timing;  // every kernel waits for its predecessor before touching memory
  if (P->xshard) {
    g_pdl = false;  // follows the caller's all-reduce
    if (P->stage_limit < 3) return CUSFFT_SUCCESS;
    if ((rc = launch_keys(P, st))) return rc;
    g_pdl = !P->timing;
    if ((rc = launch_select(P, st))) return rc;
    mark(P, 3);
  }
  if (P->stage_limit < 4) return CUSFFT_SUCCESS;
  if ((rc = launch_vote(P, st))) return rc;
  mark(P, 4);
  if (P->stage_limit < 5) return CUSFFT_SUCCESS;
  if ((rc = launch_estimate(P, st))) return rc;
  mark(P, 5);
  if (P->stage_limit < 6) return CUSFFT_SUCCESS;
  if ((rc = launch_output(P, locs, vals, st))) return rc;
  mark(P, 6);
  return CUSFFT_SUCCESS;
}

// The whole transform as two concurrent branches (graph capture only): the
// location chain (fold, FFT, cutoff, vote of loops r < L_loc) on the plan's
// high-priority capture stream, and the fold + FFT of the estimation-only
// loops on a second stream; they join before the estimation.
int launch_branched(cusfft_plan_t P, const double2* x, int64_t* locs, double2* vals) {
  cudaStream_t a = P->stream, b = P->cap_stream2;
  int rc;
  // the location fold runs alone (all of DRAM); the estimation fold then
  // overlaps the location chain's FFT, cutoff and vote
  P->cur_prio = P->prio_hi;
  if ((rc = launch_fold(P, x, 0, P->nloc_local, a, true))) return rc;
  CK(cudaEventRecord(P->ev_fork, a));
  CK(cudaStreamWaitEvent(b, P->ev_fork, 0));
  P->cur_prio = P->prio_lo;
  if ((rc = launch_fold(P, x, P->nloc_local, P->Lg, b, false))) return rc;
  if ((rc = launch_bfft(P, P->nloc_local, P->Lg, b))) return rc;
  CK(cudaEventRecord(P->ev_join, b));
  P->cur_prio = P->prio_hi;
  if ((rc = launch_bfft(P, 0, P->nloc_local, a))) return rc;
  if ((rc = launch_select(P, a))) return rc;
  if ((rc = launch_vote(P, a))) return rc;
  P->cur_prio = 0;
  CK(cudaStreamWaitEvent(a, P->ev_join, 0));
  if ((rc = launch_estimate(P, a))) return rc;
  return launch_output(P, locs, vals, a);
}

// Staged variant of the two-branch graph: the location group's phase 1 runs
// alone; then the estimation group's phase 1 (DRAM-bound, k_stage at
// stage_cps CTAs per SM) overlaps the location chain (phase 2, FFT, cutoff,
// vote: L2/latency-bound) on the high-priority stream; the estimation group's
// phase 2 and FFT follow on the second stream and join before the estimation.
int launch_branched_staged(cusfft_plan_t P, const double2* x, int64_t* locs, double2* vals) {
  cudaStream_t a = P->stream, b = P->cap_stream2;
  const auto& gl = P->groups[0];
  const auto& ge = P->groups[1];
  int rc;
  P->cur_prio = P->prio_hi;
  g_pdl = false;
  if ((rc = launch_stage1(P, gl, x, a, ZeroArgs{P->d_zero, P->nzero}))) return rc;
  CK(cudaEventRecord(P->ev_fork, a));
  CK(cudaStreamWaitEvent(b, P->ev_fork, 0));
  P->cur_prio = P->prio_lo;
  g_pdl = false;
  if ((rc = launch_stage1(P, ge, x, b, ZeroArgs{nullptr, 0}))) return rc;
  if ((rc = launch_stage2(P, ge, b, ZeroArgs{nullptr, 0}))) return rc;
  if ((rc = launch_bfft(P, ge.s0, ge.s1, b))) return rc;
  CK(cudaEventRecord(P->ev_join, b));
  P->cur_prio = P->prio_hi;
  if ((rc = launch_stage2(P, gl, a, ZeroArgs{nullptr, 0}))) return rc;
  if ((rc = launch_bfft(P, gl.s0, gl.s1, a))) return rc;
  if ((rc = launch_select(P, a))) return rc;
  if ((rc = launch_vote(P, a))) return rc;
  P->cur_prio = 0;
  CK(cudaStreamWaitEvent(a, P->ev_join, 0));
  g_pdl = false;
  if ((rc = launch_estimate(P, a))) return rc;
  g_pdl = !P->timing;
  return launch_output(P, locs, vals, a);
}

// Two branches after ONE address-ordered phase 1 of all slots (the DRAM pass
// stays whole): the location slots' phase 2, FFT pass 2, cutoff and vote on
// the high-priority stream, the estimation slots' phase 2 and FFT pass 2 on a
// second stream (filling the SMs the latency-bound chain leaves idle); they
// join before the estimation.
// stage1_outside: phase 1 was launched directly on the caller's stream just
// before this graph (so the graph's launch latency overlaps it).
int launch_branched_p2(cusfft_plan_t P, const double2* x, int64_t* locs, double2* vals, bool stage1_outside = false) {
  cudaStream_t a = P->stream, b = P->cap_stream2;
  const auto& g = P->groups[0];
  const int nl = P->nloc_local, B = (int)P->B;
  const SlotParam* sp = P->d_slots + (size_t)P->lrank * P->Lg;
  const ZeroArgs z0{nullptr, 0};
  int rc;
  // the estimation branch, forked from stream a at the current point
  auto fork = [&]() -> int {
    CK(cudaEventRecord(P->ev_fork, a));
    CK(cudaStreamWaitEvent(b, P->ev_fork, 0));
    P->cur_prio = P->prio_lo;
    g_pdl = false;
    g_p2_pad = P->est_p2_pad;
    if (g.inv)  // index staging: staging in address order, phase 2 gathers through the slot's index rows
      CK(launch_fold_fft1(P, g.staging, g.inv + (size_t)nl * P->R * B, sp + nl, P->d_u + (size_t)nl * B,
                          P->d_v + (size_t)nl * B, P->Lg - nl, z0, b, false));
    else
      CK(launch_fold_fft1(P, g.staging + (size_t)nl * P->R * B, nullptr, sp + nl, P->d_u + (size_t)nl * B,
                          P->d_v + (size_t)nl * B, P->Lg - nl, z0, b, true));
    g_p2_pad = 0;
    g_pdl = true;
    int r = launch_bfft(P, nl, P->Lg, b);
    if (r) return r;
    CK(cudaEventRecord(P->ev_join, b));
    P->cur_prio = P->prio_hi;
    // the next kernel on a keeps its programmatic edge to its predecessor on a
    // (the fork's event record adds no node): its CTAs become resident early,
    // ahead of the estimation branch's
    g_pdl = true;
    return CUSFFT_SUCCESS;
  };
  P->cur_prio = P->prio_hi;
  g_pdl = false;
  if (!stage1_outside && (rc = launch_stage1(P, g, x, a, ZeroArgs{P->d_zero, P->nzero}))) return rc;
  g_pdl = !stage1_outside;
  if (P->branch_fork == 0 && (rc = fork())) return rc;
  if (stage1_outside) g_pdl = false;  // the graph's first node on a
  CK(launch_fold_fft1(P, g.staging, g.inv, sp, P->d_u, P->d_v, nl, z0, a, g.inv == nullptr));
  g_pdl = true;
  if (P->branch_fork == 1 && (rc = fork())) return rc;
  if ((rc = launch_bfft(P, 0, nl, a))) return rc;
  g_pdl = true;
  if (P->branch_fork == 2 && (rc = fork())) return rc;
  if ((rc = launch_select(P, a))) return rc;
  g_pdl = true;
  if (P->branch_fork == 3 && (rc = fork())) return rc;
  if ((rc = launch_vote(P, a))) return rc;
  P->cur_prio = 0;
  CK(cudaStreamWaitEvent(a, P->ev_join, 0));
  g_pdl = false;
  if ((rc = launch_estimate(P, a))) return rc;
  g_pdl = true;
  return launch_output(P, locs, vals, a);
}

inline bool use_branch_p2(cusfft_plan_t P) {
  return P->branch_p2 && !P->slot_fused && P->use_graph && !P->timing && P->stage_limit == 6 && P->nloc_local > 0 &&
         P->nloc_local < P->Lg && P->staged && P->groups.size() == 1 &&
         (P->stage_scatter || P->groups[0].inv) && !P->stage_split &&
         !P->skip_stage && !P->xshard;
}

// Branched execution only inside graph capture, for full-stage runs with both
// location and estimation-only slots on this rank.
inline bool use_branches(cusfft_plan_t P) {
  return P->branched && !P->slot_fused && P->use_graph && !P->timing && P->stage_limit == 6 && P->nloc_local > 0 &&
         P->nloc_local < P->Lg && (!P->staged || (P->groups.size() == 2 && !P->stage_split && !P->skip_stage));
}

// Run `body` (which enqueues on P->stream) either directly or through a cached
// CUDA graph captured on a plan-owned stream and launched on the caller's
// stream.  In timing mode the graph also holds the stage event-record nodes.
template <class F>
int run_graphed(cusfft_plan_t P, cusfft_plan_s::GraphEntry& g_plain, cusfft_plan_s::GraphEntry& g_timed, const void* a,
                const void* b, const void* c, F&& body) {
  // Timing mode launches directly: events recorded inside a graph cannot be timed.
  if (!P->use_graph || P->timing) return body();
  (void)g_timed;
  cusfft_plan_s::GraphEntry& g = g_plain;
  if (!(g.exec && g.a == a && g.b == b && g.c == c && g.lim == P->stage_limit)) {
    if (g.exec) {
      cudaGraphExecDestroy(g.exec);
      g.exec = nullptr;
    }
    if (!P->cap_stream) {
      int lo = 0, hi = 0;
      CK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
      P->prio_lo = lo;
      P->prio_hi = hi;
      CK(cudaStreamCreateWithPriority(&P->cap_stream, cudaStreamNonBlocking, hi));   // location chain
      CK(cudaStreamCreateWithPriority(&P->cap_stream2, cudaStreamNonBlocking, lo));  // estimation folds
      CK(cudaEventCreateWithFlags(&P->ev_fork, cudaEventDisableTiming));
      CK(cudaEventCreateWithFlags(&P->ev_join, cudaEventDisableTiming));
    }
    CK(cudaStreamBeginCapture(P->cap_stream, cudaStreamCaptureModeThreadLocal));
    cudaStream_t user = P->stream;
    P->stream = P->cap_stream;
    const int rc = body();
    cudaGraph_t graph = nullptr;
    const cudaError_t ce = cudaStreamEndCapture(P->cap_stream, &graph);
    P->stream = user;
    if (rc != CUSFFT_SUCCESS) {
      if (graph) cudaGraphDestroy(graph);
      return rc;
    }
    CK(ce);
    // node priorities (location branch high, estimation branch low) are honoured only
    // with UseNodePriority (CUSFFT_NODE_PRIO=0: the launching stream's priority for all)
    const char* np = std::getenv("CUSFFT_NODE_PRIO");
    const unsigned long long iflags = (np && np[0] == '0') ? 0ull : (unsigned long long)cudaGraphInstantiateFlagUseNodePriority;
    const cudaError_t ie = cudaGraphInstantiateWithFlags(&g.exec, graph, iflags);
    cudaGraphDestroy(graph);
    CK(ie);
    g.a = a;
    g.b = b;
    g.c = c;
    g.lim = P->stage_limit;
  }
  CK(cudaGraphLaunch(g.exec, P->stream));
  return CUSFFT_SUCCESS;
}

// The cache entry for a whole-transform graph of (a, b, c) at the current stage limit.
cusfft_plan_s::GraphEntry& full_entry(cusfft_plan_t P, const void* a, const void* b, const void* c) {
  if (P->timing) return P->g_full;  // timing mode launches directly
  size_t lru = 0;
  for (size_t i = 0; i < P->g_cache.size(); ++i) {
    const auto& g = P->g_cache[i];
    if (g.exec && g.a == a && g.b == b && g.c == c && g.lim == P->stage_limit) {
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
  if (plan->split_launch && use_branch_p2(plan)) {  // phase 1 launched directly, the rest as a graph
    const double2* x = reinterpret_cast<const double2*>(d_x);
    g_pdl = false;
    plan->cur_prio = 0;
    int rc = launch_stage1(plan, plan->groups[0], x, plan->stream, ZeroArgs{plan->d_zero, plan->nzero});
    if (rc) return rc;
    return run_graphed(plan, full_entry(plan, d_x, d_locs, d_vals), plan->g_full_t, d_x, d_locs, d_vals, [&] {
      return launch_branched_p2(plan, x, d_locs, reinterpret_cast<double2*>(d_vals), true);
    });
  }
  return run_graphed(plan, full_entry(plan, d_x, d_locs, d_vals), plan->g_full_t, d_x, d_locs, d_vals, [&] {
    const double2* x = reinterpret_cast<const double2*>(d_x);
    double2* v = reinterpret_cast<double2*>(d_vals);
    if (use_branch_p2(plan)) return launch_branched_p2(plan, x, d_locs, v);
    if (use_branches(plan))
      return plan->staged ? launch_branched_staged(plan, x, d_locs, v) : launch_branched(plan, x, d_locs, v);
    int rc = launch_local(plan, x);
    if (rc) return rc;
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

const char* cusfft_strerror(int code) {
  switch (code) {
    case CUSFFT_SUCCESS: return "success";
    case CUSFFT_INVALID_N: return "n must be a power of two in [16, 2^31]";
    case CUSFFT_INVALID_B: return "B must be a power of two with 2 <= B < n";
    case CUSFFT_INVALID_K: return "need 1 <= k <= 8192 and k <= num_select <= B";
    case CUSFFT_INVALID_LOOPS: return "need 1 <= T <= L_loc <= L <= 64, L_loc <= 32 and world | L (loop sharding)";
    case CUSFFT_INVALID_PARAM: return "invalid filter or plan parameter";
    case CUSFFT_NULL_PTR: return "null pointer argument";
    case CUSFFT_ALLOC: return "device allocation failed";
    case CUSFFT_CUDA: return "CUDA runtime error (see cusfft_last_cuda_error)";
    case CUSFFT_HIT_OVERFLOW: return "more than max_hits frequencies reached the vote threshold";
    case CUSFFT_INVALID_PLAN: return "invalid or destroyed plan";
    case CUSFFT_INTERNAL: return "device-side consistency check failed";
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
  return CUSFFT_SUCCESS;
}

int cusfft_plan(cusfft_plan_t* out, int64_t n, int64_t k, int64_t B, int32_t L, const cusfft_params* p) {
  return make_plan(out, n, k, B, L, p, 0, 1);
}

int cusfft_plan_dist(cusfft_plan_t* out, int64_t n, int64_t k, int64_t B, int32_t L, const cusfft_params* p,
                     int32_t rank, int32_t world) {
  return make_plan(out, n, k, B, L, p, rank, world);
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
  return run_graphed(plan, plan->g_local, plan->g_local_t, d_x, nullptr, nullptr,
                     [&] { return launch_local(plan, reinterpret_cast<const double2*>(d_x)); });
}

int cusfft_execute_finish(cusfft_plan_t plan, int64_t* d_locs, void* d_vals) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (!d_locs || !d_vals) return CUSFFT_NULL_PTR;
  DeviceGuard g(plan->device);
  return run_graphed(plan, plan->g_finish, plan->g_finish_t, d_locs, d_vals, nullptr,
                     [&] { return launch_finish(plan, d_locs, reinterpret_cast<double2*>(d_vals)); });
}

int cusfft_execute(cusfft_plan_t plan, const void* d_x, int64_t* d_locs, void* d_vals) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (!d_x || !d_locs || !d_vals) return CUSFFT_NULL_PTR;
  if (plan->world != 1) return CUSFFT_INVALID_LOOPS;
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
  CK(cudaMemcpyAsync(plan->d_xbuf, h_x, (size_t)plan->n * 16, cudaMemcpyHostToDevice, st));
  rc = run_graphed(plan, full_entry(plan, plan->d_xbuf, plan->d_locs_buf, plan->d_vals_buf), plan->g_full_t,
                   plan->d_xbuf, plan->d_locs_buf, plan->d_vals_buf, [&] {
    if (use_branch_p2(plan)) return launch_branched_p2(plan, plan->d_xbuf, plan->d_locs_buf, plan->d_vals_buf);
    if (use_branches(plan))
      return plan->staged ? launch_branched_staged(plan, plan->d_xbuf, plan->d_locs_buf, plan->d_vals_buf)
                          : launch_branched(plan, plan->d_xbuf, plan->d_locs_buf, plan->d_vals_buf);
    int r = launch_local(plan, plan->d_xbuf);
    if (r) return r;
    return launch_finish(plan, plan->d_locs_buf, plan->d_vals_buf);
  });
  if (rc) return rc;
  CK(cudaMemcpyAsync(h_locs, plan->d_locs_buf, (size_t)plan->k * 8, cudaMemcpyDeviceToHost, st));
  CK(cudaMemcpyAsync(h_vals, plan->d_vals_buf, (size_t)plan->k * 16, cudaMemcpyDeviceToHost, st));
  return cusfft_status(plan);
}

int cusfft_exchange_buffer(cusfft_plan_t plan, void** d_buf, int64_t* bytes_per_rank) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (!d_buf || !bytes_per_rank) return CUSFFT_NULL_PTR;
  *d_buf = plan->d_records;
  *bytes_per_rank = (int64_t)plan->Lg * plan->lay.rec_bytes;
  return CUSFFT_SUCCESS;
}

int32_t cusfft_exchange_kind(cusfft_plan_t plan) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  return plan->xshard ? 1 : 0;
}

int cusfft_get_info(cusfft_plan_t plan, int64_t* info, int64_t* a, int64_t* sigma, int64_t* tau) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  if (info) {
    int64_t v[12] = {plan->n, plan->k, plan->B, plan->L, plan->w, plan->nb, plan->num, plan->Lloc, plan->T,
                     plan->max_hits, plan->sectors, plan->staged ? 1 : 0};
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
  int64_t need = 0;
  switch (what) {
    case CUSFFT_DEBUG_U: need = (int64_t)plan->Lg * B * 16; break;
    case CUSFFT_DEBUG_UHAT: need = L * B * 16; break;
    case CUSFFT_DEBUG_WINNERS: need = (int64_t)plan->Lloc * plan->Jcap * 4; break;
    case CUSFFT_DEBUG_HITS: need = H * 4; break;
    case CUSFFT_DEBUG_HIT_VALS: need = H * 16; break;
    case CUSFFT_DEBUG_PER_LOOP: need = plan->d_per_loop ? H * L * 16 : 0; break;
    case CUSFFT_DEBUG_TAPS: need = (int64_t)plan->w * 8; break;
    case CUSFFT_DEBUG_GHAT: need = (plan->nb + 1) * 16; break;
    case CUSFFT_DEBUG_NUM_HITS: need = 8; break;
    default: return CUSFFT_INVALID_PARAM;
  }
  if (!dst || cap < need || need == 0) return need;
  uint8_t* out = reinterpret_cast<uint8_t*>(dst);
  switch (what) {
    case CUSFFT_DEBUG_U:
      if (!plan->prm.debug && u_debug_only(plan)) return CUSFFT_INVALID_PARAM;  // not written
      CK(cudaMemcpy(out, plan->d_u, need, cudaMemcpyDeviceToHost));
      break;
    case CUSFFT_DEBUG_UHAT:
      for (int r = 0; r < L; ++r)
        CK(cudaMemcpy(out + (int64_t)r * B * 16, plan->d_records + (int64_t)slot_of(r) * plan->lay.rec_bytes, B * 16,
                      cudaMemcpyDeviceToHost));
      break;
    case CUSFFT_DEBUG_WINNERS:
      for (int r = 0; r < plan->Lloc; ++r) {
        const uint8_t* rec = plan->d_records + (int64_t)slot_of(r) * plan->lay.rec_bytes;
        int cnt = 0;
        CK(cudaMemcpy(&cnt, rec + plan->lay.off_cnt, 4, cudaMemcpyDeviceToHost));
        cnt = std::max(0, std::min(cnt, plan->Jcap));
        int32_t* o = reinterpret_cast<int32_t*>(out + (int64_t)r * plan->Jcap * 4);
        CK(cudaMemcpy(o, rec + plan->lay.off_J, (int64_t)cnt * 4, cudaMemcpyDeviceToHost));
        for (int j = cnt; j < plan->Jcap; ++j) o[j] = -1;
      }
      break;
    case CUSFFT_DEBUG_HITS:
      CK(cudaMemcpy(out, plan->d_hits, need, cudaMemcpyDeviceToHost));
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
      CK(cudaMemcpy(out, plan->d_taps, need, cudaMemcpyDeviceToHost));
      break;
    case CUSFFT_DEBUG_GHAT:
      CK(cudaMemcpy(out, plan->d_ghat, need, cudaMemcpyDeviceToHost));
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
  plan->timing = enable != 0;
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
    if (cudaEventElapsedTime(&t, plan->ev[i], plan->ev[i + 1]) != cudaSuccess) {
      t = -1.f;
      cudaGetLastError();  // do not leave a stale error for later launch checks
    }
    ms[i] = t;
  }
  if (cap >= 7) {
    float t = -1.f;
    if (!plan->staged || cudaEventElapsedTime(&t, plan->ev[0], plan->ev[7]) != cudaSuccess) {
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
// Reset the trace: phase slots 0, per-kernel start slots (128 + 2 id) ~0.
int cusfft_debug_trace_reset() {
  unsigned long long init[256];
  for (int i = 0; i < 256; ++i) init[i] = (i >= 128 && (i % 2) == 0) ? ~0ull : 0ull;
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpyToSymbol(g_trace, init, sizeof(init)));
  return CUSFFT_SUCCESS;
}
#endif

int32_t cusfft_launches_per_execute(cusfft_plan_t plan) {
  if (!valid_plan(plan)) return CUSFFT_INVALID_PLAN;
  const bool pass1 = plan->B1 > 1 && (!plan->fused1 || (plan->staged && plan->stage_split));
  int n = (plan->staged ? 2 * (int)plan->groups.size() : 1) /*stage + fold per group*/ + (pass1 ? 2 : 1) /*fft*/ +
          (plan->sel_slots_h.empty() ? 0 : 1) + (plan->xshard && !plan->sel_slots_h.empty() ? 1 : 0) /*keys*/ +
          3 /*vote,est,out*/;
  if (use_branch_p2(plan)) n += 2;  // phase 2 and FFT pass 2 launched per branch
  return n;
}

}  // extern "C"
