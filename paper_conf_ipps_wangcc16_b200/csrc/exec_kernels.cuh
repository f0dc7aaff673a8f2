// exec_kernels.cuh — the timed hot path:
//   k_fold      Steps 1+2  permutation + filter + fold into B buckets
//   k_fft       Step 3     batched B-point FFT (fft.cuh; one or two passes)
//   k_select    Step 4     exact top-num cutoff per location loop
//   k_vote      Step 5     reverse hash + vote
//   k_estimate  Step 6     per-loop estimates and their median
//   k_output    output     top-k hits by |val|^2, sorted by location
#pragma once
#include <cooperative_groups.h>

#include "common.cuh"
#include "fft.cuh"

namespace cusfft {

// ---------------------------------------------------------------------------
// Steps 1+2 (Alg. 1 L164-L168 semantics, Fig. 3 L187 index mapping,
// Alg. 2 L200-L226 loop partition): thread (slot s, bucket j) computes
//   u_s[j] = sum_{rr < R, i = j + rr B < w} g_i * x[(sigma_s i + tau_s) mod n]
// with the rounds accumulated in increasing i, each term one fp64 multiply and
// one fp64 add per component (no FMA contraction), i.e. Alg. 1's order.
// All RC gathers of a chunk are issued before the first add (memory-level
// parallelism); gathers use the non-coherent path without L1 allocation.
// ---------------------------------------------------------------------------
// Per-execution block zeroed by the CTAs of the first fold launch (the fold is
// memory-latency bound, so the stores are free): flags, histograms, counters.
constexpr int kMaxLoops = 64;  // L limit (plan validation)

struct ZeroArgs {
  int* p;
  int n;
};

__device__ __forceinline__ void zero_part(const ZeroArgs& z) {
  if (!z.p) return;
  const int nblk = gridDim.x * gridDim.y;
  const int blk = blockIdx.y * gridDim.x + blockIdx.x;
  const int chunk = (z.n + nblk - 1) / nblk;
  const int b = blk * chunk, e = min(z.n, b + chunk);
  for (int i = b + threadIdx.x; i < e; i += blockDim.x) z.p[i] = 0;
}

// Random 16-B gather: non-coherent path, no L1 allocation, and an L2 fetch of
// 64 B instead of the default 128-B line (halves the DRAM bytes per random
// sample; the time is bound by DRAM row activations either way, see
// scripts/probes/gather_probe.cu and DESIGN.md §6).
__device__ __forceinline__ double2 ld_gather(const double2* p) {
  double2 v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::64B.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  return v;
}

// x holds samples [xlo, xlo + xspan) of the signal (xlo = 0, xspan = n unless
// the plan is signal-sharded): a gather outside the range
// contributes nothing, so the ranks' partial buckets sum to the full fold.
template <int RC>
__global__ void __launch_bounds__(256) k_fold(const double2* __restrict__ x, const double* __restrict__ taps,
                                              const SlotParam* __restrict__ slots, double2* __restrict__ u,
                                              int B, int w, int R, uint32_t nmask, uint32_t xlo, uint32_t xspan,
                                              ZeroArgs zero) {
  pdl_wait();
  KTRACE(4);
  const int j = blockIdx.x * blockDim.x + threadIdx.x;
  const int s = blockIdx.y;
  if (blockIdx.x == 0 && blockIdx.y == 0) TRACE(0);
  zero_part(zero);
  if (j >= B) return;
  const uint32_t sigma = slots[s].sigma, tau = slots[s].tau;
  double ar = 0.0, ai = 0.0;
  for (int r0 = 0; r0 < R; r0 += RC) {
    double2 v[RC];
    double g[RC];
    bool ok[RC];
#pragma unroll
    for (int c = 0; c < RC; ++c) {
      const int i = j + (r0 + c) * B;
      const uint32_t rel = ((sigma * (uint32_t)i + tau) & nmask) - xlo;  // mod n, n | 2^32
      ok[c] = r0 + c < R && i < w && rel < xspan;
      if (ok[c]) {
        v[c] = ld_gather(x + rel);
        g[c] = __ldg(taps + i);
      }
    }
#pragma unroll
    for (int c = 0; c < RC; ++c) {
      if (ok[c]) {
        ar = __dadd_rn(ar, __dmul_rn(g[c], v[c].x));
        ai = __dadd_rn(ai, __dmul_rn(g[c], v[c].y));
      }
    }
  }
  u[(size_t)s * B + j] = make_double2(ar, ai);
  TRACE_END(1);
}

// ---------------------------------------------------------------------------
// The paper's asynchronous data layout transformation (PAPER.md:L345-L351,
// §V.A, Fig. 4) as an ablation (params.gather = 2): the fold of one loop is
// split into a remapping kernel, A'[j] = x[index(i0 + j)] for one chunk of B
// taps (chunk size B, L349), and an execution kernel that folds the chunk from
// the reordered array, u[j] += g[i0 + j] A'[j]; chunks of different loops run
// on concurrent streams.  Same per-bucket addition order as k_fold (rounds
// ascending, __dmul_rn / __dadd_rn), so u is bit-identical.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_remap(const double2* __restrict__ x, double2* __restrict__ ap,
                                               uint32_t sigma, uint32_t tau, int i0, int B, int w, uint32_t nmask) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= B) return;
  const int i = i0 + j;
  ap[j] = i < w ? ld_gather(x + ((sigma * (uint32_t)i + tau) & nmask)) : make_double2(0.0, 0.0);
}

__global__ void __launch_bounds__(256) k_remap_exec(const double2* __restrict__ ap, const double* __restrict__ taps,
                                                    double2* __restrict__ u, int i0, int B, int w) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= B) return;
  const int i = i0 + j;
  double2 acc = i0 == 0 ? make_double2(0.0, 0.0) : u[j];
  if (i < w) {
    const double g = __ldg(taps + i);
    const double2 a = ap[j];
    acc.x = __dadd_rn(acc.x, __dmul_rn(g, a.x));
    acc.y = __dadd_rn(acc.y, __dmul_rn(g, a.y));
  }
  u[j] = acc;
}

// ---------------------------------------------------------------------------
// Staged gather, phase 1: the plan sorted every (slot, tap)
// gather of this rank by address; the kernel walks them in that order, so
// DRAM rows are opened once for all loops' samples that share them (the
// random-order gather is bound by row activations), and stores each sample
// where phase 2 reads it (scatter).  x is read evict-first with 64-B L2
// fetches; the staging buffer (L2-sized) is written evict-last for phase 2.
// Also zeroes the per-execution block (first kernel of the execution).
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint64_t l2_policy_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t l2_policy_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}

// The schedule holds one word per gather, (local slot << ibits) | tap index
// i, in address order; the position sigma_s i + tau_s and phase 2's
// thread-order destination
//   (row0_s + rr) B + tile 256 + (c mod C) B1 + j1,  i = rr B + j, j = c + B2 j1,
// are recomputed here (shifts and masks; row0_s = first staging row of slot
// s, slots of a filter group have R_g rows each).
struct StagePackArgs {
  const double2* x;
  const uint32_t* code;
  double2* staging;
  const SlotParam* slots;  // local slot 0
  const uint32_t* row0;    // [nslots] first staging row of each local slot
  int total, nslots, ibits, logB, logB2, logB1, logC;
  uint32_t nmask;
  ZeroArgs zero;
  int rows;  // staging rows this launch writes into (from row 0)
};

// U: gathers in flight per thread per pass (1 at 4 CTAs of 256 per SM; U = 2, 4, 8 and 2-3 CTAs
// per SM measured equal or slower once the schedule words are prefetched).
#ifndef CUSFFT_STAGE_U
#define CUSFFT_STAGE_U 1
#endif
constexpr int kStageU = CUSFFT_STAGE_U;
template <int U>
__global__ void __launch_bounds__(256) k_stage_packed(StagePackArgs A) {
  pdl_wait();
  KTRACE(1);
  if (blockIdx.x == 0) TRACE(0);
  __shared__ uint32_t ssig[kMaxLoops], stau[kMaxLoops], srow[kMaxLoops];
  for (int i = threadIdx.x; i < A.nslots; i += blockDim.x) {
    ssig[i] = A.slots[i].sigma;
    stau[i] = A.slots[i].tau;
    srow[i] = A.row0[i];
  }
  zero_part(A.zero);
  // The staging lines are requested into L2 (evict_last) before the scattered
  // stores land on them: when they are not resident (the cold state: after
  // cudaCtxResetPersistingL2Cache or other work evicted them) every 16-B store
  // would otherwise miss on its own (phase 1 cold: 46 -> 31 µs; warm they hit,
  // +0.25 µs per transform; profiles/r02_stage_ab.md).  Fire-and-forget: the
  // gathers do not wait on them.
  {
    const int64_t lines = (int64_t)A.rows << A.logB >> 3;  // 128-B lines (8 samples each)
    const char* base = reinterpret_cast<const char*>(A.staging);
    for (int64_t l = blockIdx.x * blockDim.x + threadIdx.x; l < lines; l += gridDim.x * blockDim.x)
      asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(base + (l << 7)));
  }
  __syncthreads();
  const uint64_t pf = l2_policy_first(), pl = l2_policy_last();
  const uint32_t imask = (1u << A.ibits) - 1u;
  const uint32_t Bm = (1u << A.logB) - 1u, B2m = (1u << A.logB2) - 1u, Cm = (1u << A.logC) - 1u;
  const int T = gridDim.x * blockDim.x;
  // The schedule words are software-pipelined one pass ahead: the next pass's
  // words are requested while this pass's gathers are in flight, so no gather
  // waits on a dependent schedule load (round 1 issued word c, waited for it,
  // then gather c: U + 1 DRAM round trips per pass).
  auto ld_code = [&](int q) {
    uint32_t c;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(c) : "l"(A.code + q), "l"(pf));
    return c;
  };
  auto gather = [&](uint32_t code, double2& v) {
    const uint32_t sl = code >> A.ibits, i = code & imask;
    const double2* p = A.x + ((ssig[sl] * i + stau[sl]) & A.nmask);
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.L2::64B.v2.f64 {%0, %1}, [%2], %3;"
                 : "=d"(v.x), "=d"(v.y) : "l"(p), "l"(pf));
  };
  auto stage = [&](uint32_t code, const double2& v) {
    const uint32_t sl = code >> A.ibits, i = code & imask;
    const uint32_t rr = i >> A.logB, j = i & Bm;
    const uint32_t col = j & B2m, j1 = j >> A.logB2;
    const uint32_t dst = ((srow[sl] + rr) << A.logB) + ((col >> A.logC) << 8) + ((col & Cm) << A.logB1) + j1;
    asm volatile("st.global.L2::cache_hint.v2.f64 [%0], {%1, %2}, %3;" ::"l"(A.staging + dst), "d"(v.x), "d"(v.y),
                 "l"(pl));
  };
  const int send = A.total;
  {
    uint32_t cd[U];
    const int q00 = blockIdx.x * blockDim.x + threadIdx.x;
#pragma unroll
    for (int c = 0; c < U; ++c) {
      cd[c] = 0u;
      if (q00 + c * T < send) cd[c] = ld_code(q00 + c * T);
    }
    for (int q0 = q00; q0 < send; q0 += U * T) {
      double2 v[U];
#pragma unroll
      for (int c = 0; c < U; ++c)
        if (q0 + c * T < send) gather(cd[c], v[c]);
      uint32_t nx[U];
#pragma unroll
      for (int c = 0; c < U; ++c) {
        const int q = q0 + U * T + c * T;
        nx[c] = 0u;
        if (q < send) nx[c] = ld_code(q);
      }
#pragma unroll
      for (int c = 0; c < U; ++c) {
        if (q0 + c * T < send) stage(cd[c], v[c]);
        cd[c] = nx[c];
      }
    }
  }
  TRACE_END(6);
}

// ---------------------------------------------------------------------------
// Steps 1+2 fused with the first pass of Step 3 (four-step B = B1 x B2, B1 <=
// 256): a CTA of 256 threads folds the buckets of C = 256 / B1 whole columns
// c (j = c + B2 j1, j1 < B1) exactly as k_fold does (same per-bucket order),
// writes u (kept for parity checks), then runs the C B1-point FFTs in shared
// memory and writes v[c + B2 k1] = FFT(...)[k1] * e^{-2 pi i c k1 / B}, which
// is what the stand-alone pass 1 produces.  Taps are read from a plan-time
// permutation taps_perm[rr B + cta 256 + t] = g[j(t) + rr B] so that the tap
// loads of a CTA stay contiguous.  RC gathers per thread in flight; two CTAs
// per SM so one CTA's FFT epilogue overlaps the other's gathers.
// ---------------------------------------------------------------------------
// Direct gather from x (plans whose staging buffer would not fit L2).
template <int B1T, int RC>
__global__ void __launch_bounds__(256, 2) k_fold_fft1(const double2* __restrict__ x,
                                                      const double* __restrict__ taps_perm,
                                                      const SlotParam* __restrict__ slots,
                                                      double2* __restrict__ u, double2* __restrict__ v,
                                                      const double2* __restrict__ tw, int B, int B2,
                                                      int w, int R, uint32_t nmask, uint32_t xlo,
                                                      uint32_t xspan, ZeroArgs zero) {
  pdl_wait();
  KTRACE(2);
  constexpr int C = 256 / B1T;
  __shared__ double2 S[fft_pad_n(256)];
  __shared__ double2 twl[B1T];
  const int t = threadIdx.x;
  const int s = blockIdx.y;
  if (blockIdx.x == 0 && blockIdx.y == 0) TRACE(0);
  const int cl = t / B1T, j1 = t % B1T;
  const int c = blockIdx.x * C + cl;
  const int j = c + B2 * j1;
  zero_part(zero);
  for (int i = t; i < B1T; i += 256) twl[i] = __ldg(tw + (int64_t)i * B2);  // omega_B1^i
  const double* tp = taps_perm + (int64_t)blockIdx.x * 256 + t;
  double ar = 0.0, ai = 0.0;
  {
    const uint32_t sigma = slots[s].sigma, tau = slots[s].tau;
    for (int r0 = 0; r0 < R; r0 += RC) {
      double2 xv[RC];
      double g[RC];
      bool ok[RC];
#pragma unroll
      for (int cc = 0; cc < RC; ++cc) {
        const int i = j + (r0 + cc) * B;
        const uint32_t rel = ((sigma * (uint32_t)i + tau) & nmask) - xlo;  // mod n, n | 2^32; k_fold's range rule
        ok[cc] = r0 + cc < R && i < w && rel < xspan;
        if (ok[cc]) {
          xv[cc] = ld_gather(x + rel);
          g[cc] = __ldg(tp + (int64_t)(r0 + cc) * B);
        }
      }
#pragma unroll
      for (int cc = 0; cc < RC; ++cc) {
        if (ok[cc]) {
          ar = __dadd_rn(ar, __dmul_rn(g[cc], xv[cc].x));
          ai = __dadd_rn(ai, __dmul_rn(g[cc], xv[cc].y));
        }
      }
    }
  }
  S[fft_pad(cl * B1T + j1)] = make_double2(ar, ai);
  __syncthreads();
  // u and v hold the CTA's C columns at stride B2: write column-adjacent
  // elements from neighbouring threads (full 32-B sectors when C >= 2)
  const int wc = t % C, wj = t / C;  // writer's (column, row)
  const size_t wpos = (size_t)s * B + (size_t)blockIdx.x * C + wc + (size_t)B2 * wj;
  if (u) u[wpos] = S[fft_pad(wc * B1T + wj)];  // the fold output itself: debug plans only
  __syncthreads();
  fft_smem<B1T, 256, 256, true>(S, twl, B1T);
  // v = FFT result times omega_B^(c k1); the writer's own twiddle
  const double2 wv = __ldg(tw + (((int64_t)(blockIdx.x * C + wc) * wj) & (B - 1)));
  v[wpos] = cmul(S[fft_pad(wc * B1T + wj)], wv);
  TRACE_END(1);
}

// ---------------------------------------------------------------------------
// Phase 2 of the scatter-staged fold with bulk copies: a CTA
// owns one tile of 256 buckets of `spc` consecutive slots of one filter.  Its
// taps (R per thread) are loaded once and serve every slot; each slot's R rows
// of 256 staged samples (row rr = staging[(s R + rr) B + tile 256 ...], 4 KB
// each, already in this kernel's thread order) are moved to shared memory by
// the bulk-copy engine onto an mbarrier, double-buffered so the next slot's
// rows stream in while this one is folded.  Per slot exactly k_fold_fft1's
// arithmetic: rounds accumulated in Alg. 1's order (fp64 mul + add per
// component), u written (debug plans), the C columns' B1-point FFTs in shared
// memory, v = FFT x omega_B^(c k1).  The consumed staging lines stay in L2
// (the persisting set-aside): the next execution's phase-1 stores then hit
// valid lines.
// ---------------------------------------------------------------------------
// RMAX: taps held in registers (8 when R <= 8, else 16; rounds beyond reload theirs).
template <int B1T, int RMAX>
__global__ void __launch_bounds__(256, 2) k_fold_fft1_tma(const double2* __restrict__ staging,
                                                          const double* __restrict__ taps_perm,
                                                          double2* __restrict__ u, double2* __restrict__ v,
                                                          const double2* __restrict__ tw, int B, int B2, int w, int R,
                                                          int nslots, int spc, ZeroArgs zero) {
  pdl_wait();
  KTRACE(2);
  constexpr int C = 256 / B1T;
  extern __shared__ __align__(128) double2 Tile[];  // [nbuf][R][256]
  __shared__ double2 S[fft_pad_n(256)];
  __shared__ double2 twl[B1T];
  __shared__ __align__(8) uint64_t bar[2];
  const int t = threadIdx.x;
  const int s0 = blockIdx.y * spc;
  const int ns = min(spc, nslots - s0);
  if (blockIdx.x == 0 && blockIdx.y == 0) TRACE(0);
  const double2* src0 = staging + (int64_t)s0 * R * B + (int64_t)blockIdx.x * 256;
  const uint32_t bytes = (uint32_t)R * 4096u;
  // thread 0: slot i's R rows into buffer i & 1 (its barrier's next phase)
  auto issue = [&](int i) {
    uint64_t* b = bar + (i & 1);
    mbar_expect_tx(b, bytes);
    const uint64_t pol = l2_policy_first();
    const double2* src = src0 + (int64_t)i * R * B;
    double2* dst = Tile + (size_t)(i & 1) * R * 256;
    for (int rr = 0; rr < R; ++rr) bulk_g2s(dst + rr * 256, src + (int64_t)rr * B, 4096u, b, pol);
  };
  if (t == 0) {
    mbar_init(bar, 1);
    mbar_init(bar + 1, 1);
    issue(0);
    if (ns > 1) issue(1);
  }
  zero_part(zero);
  const int cl = t / B1T, j1 = t % B1T;
  const int c = blockIdx.x * C + cl;
  const int j = c + B2 * j1;
  for (int i = t; i < B1T; i += 256) twl[i] = __ldg(tw + (int64_t)i * B2);  // omega_B1^i
  const double* tp = taps_perm + (int64_t)blockIdx.x * 256 + t;
  double g[RMAX];
#pragma unroll
  for (int rr = 0; rr < RMAX; ++rr) g[rr] = (rr < R && j + rr * B < w) ? __ldg(tp + (int64_t)rr * B) : 0.0;
  const int wc = t % C, wj = t / C;  // writer's (column, row)
  const double2 wv = __ldg(tw + (((int64_t)(blockIdx.x * C + wc) * wj) & (B - 1)));
  __syncthreads();  // barrier init visible to every thread
#ifdef CUSFFT_TRACE
  const long long fc0 = clock64();
  const int fsel = blockIdx.y * gridDim.x + blockIdx.x;
  if (t == 0) atomicMax(&g_trace[112 + (zero.p != nullptr)], gtimer());  // latest CTA start (per launch)
#endif
  for (int i = 0; i < ns; ++i) {
    const double2* T = Tile + (size_t)(i & 1) * R * 256;
    mbar_wait(bar + (i & 1), (uint32_t)((i >> 1) & 1));
#ifdef CUSFFT_TRACE
    if (i == 0) CTRACE_MAX(114, clock64() - fc0);  // first slot's rows landed
    const long long fc1 = clock64();
#endif
    double ar = 0.0, ai = 0.0;
#pragma unroll
    for (int rr = 0; rr < RMAX; ++rr) {
      if (rr < R && j + rr * B < w) {
        const double2 q = T[rr * 256 + t];
        ar = __dadd_rn(ar, __dmul_rn(g[rr], q.x));
        ai = __dadd_rn(ai, __dmul_rn(g[rr], q.y));
      }
    }
    for (int rr = RMAX; rr < R; ++rr) {  // R > 16 (small tolerance / Gaussian filters)
      if (j + rr * B < w) {
        const double2 q = T[rr * 256 + t];
        const double gg = __ldg(tp + (int64_t)rr * B);
        ar = __dadd_rn(ar, __dmul_rn(gg, q.x));
        ai = __dadd_rn(ai, __dmul_rn(gg, q.y));
      }
    }
    S[fft_pad(cl * B1T + j1)] = make_double2(ar, ai);
    __syncthreads();  // every thread is done with buffer i & 1
    if (t == 0 && i + 2 < ns) issue(i + 2);
    const size_t wpos = (size_t)(s0 + i) * B + (size_t)blockIdx.x * C + wc + (size_t)B2 * wj;
    if (u) u[wpos] = S[fft_pad(wc * B1T + wj)];  // the fold output itself: debug plans only
    __syncthreads();
    fft_smem<B1T, 256, 256, true>(S, twl, B1T);
    v[wpos] = cmul(S[fft_pad(wc * B1T + wj)], wv);
    __syncthreads();  // S is rewritten by the next slot
#ifdef CUSFFT_TRACE
    CTRACE_MAX(115, clock64() - fc1);  // one slot's fold + column FFT
#endif
  }
#ifdef CUSFFT_TRACE
  CTRACE_MAX(116, clock64() - fc0);
  (void)fsel;
#endif
  TRACE_END(1);
}

// ---------------------------------------------------------------------------
// Phase 2, multi-slot form: a CTA owns one tile of 256 buckets (C = 256 / B1
// columns) of up to NSMAX slots of one filter.  Thread t folds bucket
// (c, j1) of every slot; its R staged samples of each slot (row rr element t
// of the tile: exactly the ones it folds) are copied to shared memory by
// cp.async, NBUF slots in flight (a per-thread ring: no barrier between
// slots).  After the last slot the CTA runs the column FFTs of ALL its slots
// at once (NSMAX C sequences of B1) and writes v.  Per slot the arithmetic is
// k_fold_fft1_tma's (Alg. 1 order).  Dynamic smem: fold_ms_smem_bytes.
// ---------------------------------------------------------------------------
template <int B1T, int NSMAX, int NBUF, int RMAX>
__host__ __device__ constexpr int fold_ms_smem_bytes() {
  return NBUF * RMAX * 256 * 16 + fft_pad_n(NSMAX * 256) * 16 + B1T * 16;
}

__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

template <int B1T, int NSMAX, int NBUF, int RMAX>
__global__ void __launch_bounds__(256, 1) k_fold_fft1_ms(const double2* __restrict__ staging,
                                                         const double* __restrict__ taps_perm,
                                                         double2* __restrict__ u, double2* __restrict__ v,
                                                         const double2* __restrict__ tw, int B, int B2, int w, int R,
                                                         int nslots, ZeroArgs zero) {
  pdl_wait();
  KTRACE(2);
  constexpr int C = 256 / B1T;
  constexpr int E = NSMAX * 256;
  extern __shared__ __align__(16) uint8_t msm[];
  double2* Ring = reinterpret_cast<double2*>(msm);  // [NBUF][RMAX][256]
  double2* S = Ring + NBUF * RMAX * 256;            // fft_pad_n(E)
  double2* twl = S + fft_pad_n(E);                  // B1T
  const int t = threadIdx.x;
  const int s0 = blockIdx.y * NSMAX;
  const int ns = min(NSMAX, nslots - s0);
  if (blockIdx.x == 0 && blockIdx.y == 0) TRACE(0);
  const int cl = t / B1T, j1 = t % B1T;
  const int c = blockIdx.x * C + cl;
  const int j = c + B2 * j1;
  const double2* src0 = staging + (int64_t)s0 * R * B + (int64_t)blockIdx.x * 256 + t;
  auto issue = [&](int i) {  // my R samples of slot i into ring slot i mod NBUF
    if (i < ns) {
      double2* dst = Ring + (i % NBUF) * RMAX * 256 + t;
      const double2* src = src0 + (int64_t)i * R * B;
#pragma unroll
      for (int rr = 0; rr < RMAX; ++rr)
        if (rr < R && j + rr * B < w) cp_async16(dst + rr * 256, src + (int64_t)rr * B);
    }
    cp_async_commit();  // (empty groups keep the count uniform)
  };
#pragma unroll
  for (int i = 0; i < NBUF; ++i) issue(i);
  zero_part(zero);
  for (int i = t; i < B1T; i += 256) twl[i] = __ldg(tw + (int64_t)i * B2);  // omega_B1^i
  const double* tp = taps_perm + (int64_t)blockIdx.x * 256 + t;
  double g[RMAX];
#pragma unroll
  for (int rr = 0; rr < RMAX; ++rr) g[rr] = (rr < R && j + rr * B < w) ? __ldg(tp + (int64_t)rr * B) : 0.0;
  const int wc = t % C, wj = t / C;  // writer's (column, row)
  const double2 wv = __ldg(tw + (((int64_t)(blockIdx.x * C + wc) * wj) & (B - 1)));
  for (int i = 0; i < ns; ++i) {
    cp_async_wait<NBUF - 1>();  // slot i's group (my own copies: no barrier)
    const double2* T = Ring + (i % NBUF) * RMAX * 256 + t;
    double ar = 0.0, ai = 0.0;
#pragma unroll
    for (int rr = 0; rr < RMAX; ++rr) {
      if (rr < R && j + rr * B < w) {
        const double2 q = T[rr * 256];
        ar = __dadd_rn(ar, __dmul_rn(g[rr], q.x));
        ai = __dadd_rn(ai, __dmul_rn(g[rr], q.y));
      }
    }
    S[fft_pad(i * 256 + cl * B1T + j1)] = make_double2(ar, ai);
    issue(i + NBUF);  // into the ring slot just consumed (by this thread only)
  }
  cp_async_wait<0>();
  __syncthreads();
  if (u)  // the fold output itself: debug plans only
    for (int i = 0; i < ns; ++i)
      u[(size_t)(s0 + i) * B + (size_t)blockIdx.x * C + wc + (size_t)B2 * wj] = S[fft_pad(i * 256 + wc * B1T + wj)];
  fft_smem<B1T, E, 256, true>(S, twl, B1T);
  for (int i = 0; i < ns; ++i)
    v[(size_t)(s0 + i) * B + (size_t)blockIdx.x * C + wc + (size_t)B2 * wj] =
        cmul(S[fft_pad(i * 256 + wc * B1T + wj)], wv);
  TRACE_END(1);
}

// ---------------------------------------------------------------------------
// Record layout of one slot in the exchange buffer:
//   [u^ : B x double2][bitmap : B/32 x u32][count : int32][J : Jcap x int32],
//   256-B aligned; Jcap = num (B in THRESHOLD mode).
// ---------------------------------------------------------------------------
struct RecLayout {
  int64_t rec_bytes, off_bitmap, off_cnt, off_J;
};


struct KeysSrc {
  const uint64_t* keys;
  __device__ __forceinline__ void get(int i, uint64_t& hi, uint32_t& lo) const {
    hi = keys[i];
    lo = ~(uint32_t)i;
  }
};

struct PairSrc {  // (key, index) pairs; the index is the tie-break
  const uint64_t* keys;
  const int* idx;
  __device__ __forceinline__ void get(int i, uint64_t& hi, uint32_t& lo) const {
    hi = keys[i];
    lo = ~(uint32_t)idx[i];
  }
};

// Two-level top-K selection shared by the cutoff and the output selection
// (blockDim.x == 1024).  Level 0: the producer kernel counted the items per
// top digit (pass 0) into `ghist` (global, reset here).  One pass over the N
// items (key(i), tie(i)) then accepts every item above the boundary digit
// (on_sel(i)), keeps the boundary bin's items as smem candidates and counts
// their pass-1 digits; a radix select among the candidates (usually one
// histogram scan) finishes the job.  Falls back to a full radix select when the
// boundary bin holds more than `cap` items.  hist: 4096 u32 smem; sm >= 64 ints.
template <class KeyAt, class OnSel>
__device__ void select_topk(int N, int K, uint32_t* ghist, KeyAt key_at, OnSel on_sel, uint64_t* ckey, int* cidx,
                            int cap, uint32_t* hist, int* sm) {
  const int tid = threadIdx.x;
  const BinPick b0 = pick_bin(ghist, K, sm);
  for (int i = tid; i < 4096; i += 1024) hist[i] = 0;
  if (tid == 0) sm[40] = 0;
  __syncthreads();
  const uint32_t d0 = (uint32_t)b0.d;
  const int k2 = K - b0.above;  // 1 <= k2 <= b0.cnt
  const bool whole = (k2 == b0.cnt);
  const int shift1 = pass_shift(1);
  for (int i0 = 0; i0 < N; i0 += 8 * 1024) {
    uint64_t kb[8];
    uint32_t tb[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int i = i0 + u * 1024 + tid;
      if (i < N) key_at(i, kb[u], tb[u]);
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int i = i0 + u * 1024 + tid;
      if (i >= N) continue;
      const uint32_t d = (uint32_t)(kb[u] >> 51) & 0xFFFu;
      if (d > d0 || (d == d0 && whole)) {
        on_sel(i);
      } else if (d == d0) {
        const int pos = atomicAdd(&sm[40], 1);
        if (pos < cap) {
          ckey[pos] = kb[u];
          cidx[pos] = i;
        }
        atomicAdd(&hist[digit96(kb[u], ~tb[u], shift1)], 1u);
      }
    }
  }
  __syncthreads();
  if (whole) return;
  const int nc = sm[40];
  Prefix96 p{0, 0, 0, 0};
  or96(p.phi, p.plo, d0, pass_shift(0));
  or96(p.mhi, p.mlo, 0xFFFu, pass_shift(0));
  if (nc <= 1024 && nc <= cap) {  // few candidates: exact rank counting, one pass
    uint64_t mk = 0;
    uint32_t mt = 0;
    if (tid < nc) {
      mk = ckey[tid];
      uint64_t kk;
      key_at(cidx[tid], kk, mt);
      cidx[cap - 1 - tid] = (int)mt;  // tie values, stored from the top of cidx
    }
    __syncthreads();
    if (tid < nc) {
      int rank = 0;  // preferred: larger key, or equal key and smaller tie value
      for (int c = 0; c < nc; ++c) {
        const uint64_t kc = ckey[c];
        rank += (kc > mk) || (kc == mk && (uint32_t)cidx[cap - 1 - c] < mt);
      }
      if (rank < k2) on_sel(cidx[tid]);
    }
    __syncthreads();
  } else if (nc <= cap) {
    struct CandSrc {
      const uint64_t* k;
      const int* c;
      KeyAt ka;
      __device__ __forceinline__ void get(int j, uint64_t& hi, uint32_t& lo) const {
        uint32_t t;
        uint64_t kk;
        ka(c[j], kk, t);
        hi = k[j];
        lo = ~t;
      }
    };
    p = block_radix_select(CandSrc{ckey, cidx, key_at}, nc, k2, hist, sm, 1, p, true);
    for (int c = tid; c < nc; c += 1024) {
      uint64_t kk;
      uint32_t t;
      key_at(cidx[c], kk, t);
      if (ge96(p, kk, ~t)) on_sel(cidx[c]);
    }
  } else {  // crowded boundary bin: radix over all items matching the level-0 digit
    struct AllSrc {
      KeyAt ka;
      __device__ __forceinline__ void get(int j, uint64_t& hi, uint32_t& lo) const {
        uint32_t t;
        ka(j, hi, t);
        lo = ~t;
      }
    };
    p = block_radix_select(AllSrc{key_at}, N, k2, hist, sm, 1, p, true);
    for (int i = tid; i < N; i += 1024) {
      uint64_t kk;
      uint32_t t;
      key_at(i, kk, t);
      if (((kk >> 51) & 0xFFFu) == d0 && ge96(p, kk, ~t)) on_sel(i);
    }
  }
  __syncthreads();
}

// ---------------------------------------------------------------------------
// Step 4 (L89, Alg. 3; the linear-time selection of §V.B,
// made exact): J_r = the num buckets of largest |u^|^2 = re*re + im*im, ties
// to the smaller bucket, as a bitmap and an ascending list.
// Grid: S CTAs of 256 threads per location slot of this rank.  Level 0 (the
// top 12 key bits below the sign) was counted by the FFT epilogue; every CTA
// reads it, finds the boundary digit d0, and scans B/S keys, one warp per 32
// keys: a ballot of "digit > d0" is the bitmap word; boundary-bin keys go to a
// per-loop global candidate list and their next 12 bits to a level-1
// histogram.  The last CTA of the loop (threadfence + counter) resolves the
// boundary bin exactly (radix select from pass 1), ORs those bits in, resets
// the loop's counters and histograms, and writes the ascending winner list.
// ---------------------------------------------------------------------------
constexpr int kSelCap = 4096;
constexpr int kSelNT = 256;

constexpr int kMaxSel = 32;  // location loops per plan (kMaxLoc)

struct SelArgs {
  uint8_t* recs[kMaxSel];  // record of each location slot of this rank (by value)
  RecLayout lay;
  int B, num;
  int threshold_mode;  // Alg. 6: keep every key >= thr_key, no selection
  uint64_t thr_key;    // bits of the |u^|^2 threshold
  const uint64_t* keys;  // [n_sel][B]
  uint32_t* hist0;       // [n_sel][4096] (FFT epilogue)
  int* status;
  // optional (single-rank plans with every location loop selected here): the
  // vote table of k_tail (element b = bucket b, bit q = kept in location loop
  // q, selection index == vote index), ORed in by the cluster cutoff; zeroed
  // per execution
  uint32_t* pk;
  int pk_esz;      // bytes per pk element (1 / 2 / 4: L_loc <= 8 / 16 / 32)
  // optional (shard_mode 2): where selection i writes its candidate record
  // (bitmap | count | J with the record's relative offsets) instead of its
  // record, i.e. this rank's slice of the candidate all-gather buffer
  uint8_t* cout[kMaxSel];
};

struct SelOut {
  uint32_t* bitmap;
  int* cnt;
  int* J;
};
__device__ __forceinline__ SelOut sel_out(const SelArgs& A, int sel, uint8_t* rec) {
  if (uint8_t* c = A.cout[sel])
    return {reinterpret_cast<uint32_t*>(c), reinterpret_cast<int*>(c + (A.lay.off_cnt - A.lay.off_bitmap)),
            reinterpret_cast<int*>(c + (A.lay.off_J - A.lay.off_bitmap))};
  return {reinterpret_cast<uint32_t*>(rec + A.lay.off_bitmap), reinterpret_cast<int*>(rec + A.lay.off_cnt),
          reinterpret_cast<int*>(rec + A.lay.off_J)};
}

struct GKeySrc {
  const uint64_t* keys;
  __device__ __forceinline__ void get(int i, uint64_t& hi, uint32_t& lo) const {
    hi = __ldcg(keys + i);
    lo = ~(uint32_t)i;
  }
};

// Cutoff keys of the location loops from the summed bucket spectra
// (signal-sharded plans only, after the all-reduce; otherwise FFT pass 2
// emits them): key = bits(|u^|^2) and the 4096-bin top-digit histogram,
// exactly as the FFT epilogue (fft.cuh) computes them.
struct KeysArgs {
  const double2* rec[kMaxSel];  // u^ of selection index i (record start)
  uint64_t* keys;               // [n_sel][B]
  uint32_t* hist;               // [n_sel][4096]
  int B;
};

__global__ void __launch_bounds__(256) k_keys(KeysArgs A) {
  pdl_wait();
  KTRACE(7);
  __shared__ uint32_t sh[4096];
  const int i = blockIdx.y;
  for (int t = threadIdx.x; t < 4096; t += 256) sh[t] = 0;
  __syncthreads();
  const double2* u = A.rec[i];
  for (int p = blockIdx.x * 256 + threadIdx.x; p < A.B; p += gridDim.x * 256) {
    const double2 v = __ldcg(u + p);
    const uint64_t key = (uint64_t)__double_as_longlong(__dadd_rn(__dmul_rn(v.x, v.x), __dmul_rn(v.y, v.y)));
    A.keys[(int64_t)i * A.B + p] = key;
    atomicAdd(&sh[(uint32_t)(key >> 51) & 0xFFFu], 1u);
  }
  __syncthreads();
  for (int t = threadIdx.x; t < 4096; t += 256)
    if (sh[t]) atomicAdd(&A.hist[(int64_t)i * 4096 + t], sh[t]);
}

// ---------------------------------------------------------------------------
// Step 4, single-CTA form (B <= kSel1MaxB, the common case): one CTA of 1024
// threads per location slot does the whole exact selection in shared memory.
// Level 0 comes from the FFT epilogue's histogram; one pass over the keys
// (8 chunks of 1024 in flight) writes the bitmap words by ballot and appends
// boundary-bin candidates to shared memory (warp-aggregated); the boundary is
// resolved by rank counting (nc <= 256) or a radix select over the candidates
// (or over all keys of the bin when they overflow kSelCap); then the bitmap
// and the ascending winner list go out.  Same result as k_select.
// Dynamic smem: 4096 u32 + 64 int + kSelCap (u64 + int) + ceil(B/32) u32.
// ---------------------------------------------------------------------------
// Warp-parallel rank of candidate (mk, mi) among n (key, index) pairs in
// shared memory: how many are preferred to it (larger key, or equal key and
// smaller bucket).  Lanes split the pairs; one ballot per 32.
__device__ __forceinline__ int warp_rank(const uint64_t* ck, const int* ci, int n, uint64_t mk, int mi) {
  const int lane = threadIdx.x & 31;
  int rank = 0;
  for (int c0 = 0; c0 < n; c0 += 32) {
    const int c = c0 + lane;
    bool pref = false;
    if (c < n) {
      const uint64_t kc = ck[c];
      pref = (kc > mk) | ((kc == mk) & (ci[c] < mi));
    }
    rank += __popc(__ballot_sync(kFull, pref));
  }
  return rank;
}

constexpr int kSel1MaxB = 65536;

// k_tail's vote table (element b, pk_esz bytes = bucket b; bit sel = kept in
// location loop sel): OR in the 32 buckets from b0 of one bitmap word.
__device__ __forceinline__ void pk_or_word(const SelArgs& A, int sel, uint32_t bits, int64_t b0) {
  if (!bits) return;
  if (A.pk_esz == 1) {  // 4 buckets per u32: spread each nibble of bits over 4 bytes
    uint32_t* dst = A.pk + b0 / 4;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const uint32_t nib = (bits >> (4 * j)) & 0xFu;
      if (nib) atomicOr(dst + j, ((nib * 0x00204081u) & 0x01010101u) << sel);
    }
  } else {
    for (uint32_t bb = bits; bb; bb &= bb - 1) {
      const int64_t bkt = b0 + __ffs(bb) - 1;
      const int per = 4 / A.pk_esz;  // buckets per u32 word
      atomicOr(A.pk + bkt / per, (1u << sel) << (8 * A.pk_esz * (int)(bkt % per)));
    }
  }
}

// The whole single-CTA selection of slot `sel` (blockDim 1024); write_pk: also
// OR the winners into k_tail's vote table (when called as a cluster cutoff's fallback).
__device__ __forceinline__ void select1_body(const SelArgs& A, int sel, uint8_t* smem, bool write_pk) {
  uint32_t* hist = reinterpret_cast<uint32_t*>(smem);
  int* sm = reinterpret_cast<int*>(smem + 4096 * 4);
  uint64_t* skey = reinterpret_cast<uint64_t*>(smem + 4096 * 4 + 64 * 4);
  int* sidx = reinterpret_cast<int*>(skey + kSelCap);
  uint32_t* sbits = reinterpret_cast<uint32_t*>(sidx + kSelCap);
  const int tid = threadIdx.x, lane = tid & 31;
  const int B = A.B;
  uint8_t* rec = A.recs[sel];
  const uint64_t* keys = A.keys + (int64_t)sel * B;
  const int words = (B + 31) >> 5;
  if (sel == 0) TRACE(10);
  BinPick b0{0, 0, 0};
  if (!A.threshold_mode) b0 = pick_bin<1024>(A.hist0 + (int64_t)sel * 4096, A.num, sm);
  const uint32_t d0 = (uint32_t)b0.d;
  const int k2 = A.num - b0.above;
  const bool whole = A.threshold_mode || (k2 == b0.cnt);
  if (tid == 0) sm[41] = 0;
  __syncthreads();
  if (sel == 0) TRACE(11);
  const unsigned lt = (1u << lane) - 1u;
  for (int c0 = 0; c0 < B; c0 += 8 * 1024) {
    uint64_t kb[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int i = c0 + u * 1024 + tid;
      kb[u] = i < B ? __ldg(keys + i) : 0ull;
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int i = c0 + u * 1024 + tid;
      if (c0 + u * 1024 >= B) break;
      const uint32_t d = (uint32_t)(kb[u] >> 51) & 0xFFFu;
      const bool take = i < B && (A.threshold_mode ? kb[u] >= A.thr_key : (d > d0 || (d == d0 && whole)));
      const bool cand = i < B && !A.threshold_mode && d == d0 && !whole;
      const uint32_t word = __ballot_sync(kFull, take);
      if (lane == 0 && (i >> 5) < words) sbits[i >> 5] = word;
      const unsigned cm = __ballot_sync(kFull, cand);
      if (cm) {
        int base = 0;
        if (lane == __ffs(cm) - 1) base = atomicAdd(&sm[41], __popc(cm));
        base = __shfl_sync(kFull, base, __ffs(cm) - 1);
        if (cand) {
          const int pos = base + __popc(cm & lt);
          if (pos < kSelCap) {
            skey[pos] = kb[u];
            sidx[pos] = i;
          }
        }
      }
    }
  }
  __syncthreads();
  if (sel == 0) TRACE(12);
#ifdef CUSFFT_TRACE
  if (tid == 0 && sel < 16) g_trace[96 + sel] = (unsigned long long)sm[41] | ((unsigned long long)whole << 32);
#endif
  if (!whole) {
    const int nc = sm[41];
    Prefix96 p{0, 0, 0, 0};
    or96(p.phi, p.plo, d0, pass_shift(0));
    or96(p.mhi, p.mlo, 0xFFFu, pass_shift(0));
    if (nc <= 256) {  // few candidates: exact rank counting, warp per candidate
      for (int j = tid >> 5; j < nc; j += 32) {
        const int mi = sidx[j];
        const int rank = warp_rank(skey, sidx, nc, skey[j], mi);
        if (lane == 0 && rank < k2) atomicOr(&sbits[mi >> 5], 1u << (mi & 31));
      }
    } else if (nc <= kSelCap) {
      p = block_radix_select<PairSrc, 1024>(PairSrc{skey, sidx}, nc, k2, hist, sm, 1, p, false);
      for (int c = tid; c < nc; c += 1024)
        if (ge96(p, skey[c], ~(uint32_t)sidx[c])) atomicOr(&sbits[sidx[c] >> 5], 1u << (sidx[c] & 31));
    } else {  // crowded boundary bin: radix over every key of the bin
      p = block_radix_select<GKeySrc, 1024>(GKeySrc{keys}, B, k2, hist, sm, 1, p, false);
      for (int i = tid; i < B; i += 1024) {
        const uint64_t kk = __ldcg(keys + i);
        if (((kk >> 51) & 0xFFFu) == d0 && ge96(p, kk, ~(uint32_t)i)) atomicOr(&sbits[i >> 5], 1u << (i & 31));
      }
    }
  }
  __syncthreads();
  if (sel == 0) TRACE(13);
  // bitmap out + ascending winner list (thread t owns words [t wpt, (t+1) wpt))
  const SelOut so = sel_out(A, sel, rec);
  uint32_t* bitmap = so.bitmap;
  int* J = so.J;
  for (int w = tid; w < words; w += 1024) {
    bitmap[w] = sbits[w];
    if (write_pk && A.pk) pk_or_word(A, sel, sbits[w], (int64_t)w * 32);
  }
  const int wpt = (words + 1023) / 1024;
  int cnt = 0;
  for (int w = tid * wpt; w < min(words, (tid + 1) * wpt); ++w) cnt += __popc(sbits[w]);
  int total;
  int pos = block_excl_scan<1024>(cnt, &total, sm);
  for (int w = tid * wpt; w < min(words, (tid + 1) * wpt); ++w) {
    uint32_t bits = sbits[w];
    while (bits) {
      const int b = __ffs(bits) - 1;
      bits &= bits - 1;
      J[pos++] = w * 32 + b;  // pos < total <= Jcap
    }
  }
  if (tid == 0) {
    *so.cnt = total;
    if (!A.threshold_mode && total != A.num) atomicOr(A.status + 1, 1);
  }
  if (sel == 0) TRACE(14);
}

__global__ void __launch_bounds__(1024) k_select1(SelArgs A) {
  pdl_wait();
  KTRACE(8);
  extern __shared__ __align__(16) uint8_t smem[];
  select1_body(A, blockIdx.x, smem, false);
}

// ---------------------------------------------------------------------------
// Step 4, cluster form (default for 256 <= B <= 65536): a cluster of kSelCL
// CTAs per location slot, CTA r owning keys [r B/kSelCL, (r+1) B/kSelCL) and
// level-0 bins [r 4096/kSelCL, ...).  Distributed shared memory replaces the
// global candidate list and the last-CTA hand-off of k_select:
//   1. each CTA sums its bin slice; cluster barrier
//   2. the CTA holding the boundary bin finds d0 (block scan); barrier
//   3. every CTA classifies its keys: bitmap words by ballot in its own smem,
//      boundary-bin candidates appended to CTA 0's smem (remote atomics),
//      its "take" count to CTA 0; barrier
//   4. CTA 0 resolves the boundary exactly (rank counting, or radix over the
//      candidates / over all keys of the bin if they overflowed), ORs the
//      winners' bits into the owners' smem words, hands out J offsets; barrier
//   5. every CTA writes its bitmap words and its part of the ascending J.
// Same result as k_select / k_select1.
// ---------------------------------------------------------------------------
constexpr int kSelCL = 8;     // CTAs per cluster (portable maximum)
constexpr int kSelCNT = 256;  // threads per CTA

struct SelClusterSmem {
  uint32_t hist[4096];          // radix scratch
  int sm[64];
  uint64_t ckey[kSelCap];       // candidates (appended into CTA 0, copied by every CTA)
  int cidx[kSelCap];
  int ncand;                    // candidate counter (CTA 0)
  int part[kSelCL];             // bin-slice totals (pushed to every CTA)
  int pick[3];                  // d0, above, cnt (pushed by the boundary CTA)
  int cnt[kSelCL];              // final winners per CTA (pushed to every CTA)
};

// Step 5 of the cluster selection: this CTA's bitmap words, its vote-table
// bits, its part of the ascending J (from position pos) and the count.
template <int NT = kSelCNT>
__device__ __forceinline__ void select_cluster_write(const SelArgs& A, uint8_t* rec, const uint32_t* sbits, int sel,
                                                     int r, int wpc, int wpt, int k0, int pos, int total) {
  const int tid = threadIdx.x;
  const SelOut so = sel_out(A, sel, rec);
  uint32_t* bitmap = so.bitmap + r * wpc;
  int* J = so.J;
  for (int w = tid; w < wpc; w += NT) bitmap[w] = sbits[w];
  if (A.pk)  // k_tail's vote table
    for (int w = tid; w < wpc; w += NT) pk_or_word(A, sel, sbits[w], (int64_t)(r * wpc + w) * 32);
  for (int w = tid * wpt; w < min(wpc, (tid + 1) * wpt); ++w) {
    uint32_t bits = sbits[w];
    while (bits) {
      const int b = __ffs(bits) - 1;
      bits &= bits - 1;
      J[pos++] = k0 + w * 32 + b;
    }
  }
  if (r == 0 && tid == 0) {
    *so.cnt = total;
    if (!A.threshold_mode && total != A.num) atomicOr(A.status + 1, 1);
  }
}

// Fast form of the cluster selection (EXACT mode), one cluster barrier:
//   1. every CTA reads the whole 4096-bin level-0 histogram and finds the
//      boundary digit d0 itself (block scan, no exchange);
//   2. classifies its keys (bitmap words by ballot), counts the keys taken
//      outright and pushes that count and its boundary-bin candidates to
//      every CTA of the cluster (remote stores);
//   3. one cluster barrier; then every CTA holds every candidate and every
//      take count: it ranks all candidates (ties to the smaller bucket), so it
//      knows every CTA's final count (its J offset) without another round.
// Returns false (uniformly over the cluster, after the barrier) when some CTA
// holds more than kSelFastCap candidates: the caller then runs the general form.
constexpr int kSelFastCap = 64;
struct SelFastSmem {
  int sm[64];
  int take[kSelCL];                     // pushed: keys taken outright by CTA c
  int ncand[kSelCL];                    // pushed: boundary candidates of CTA c
  uint64_t ckey[kSelCL][kSelFastCap];   // pushed: candidates of CTA c
  int cidx[kSelCL][kSelFastCap];
  uint64_t fkey[kSelCL * kSelFastCap];  // local: all candidates, flat
  int fidx[kSelCL * kSelFastCap];
  int wins[kSelCL];                     // local: winners per owner CTA
  int lkey_n;                           // local: my candidates
  int pick[3];                          // local: d0, above, cnt
};

static_assert(sizeof(SelFastSmem) <= sizeof(SelClusterSmem), "fast selection smem must fit the general layout");
__device__ __forceinline__ bool select_cluster_fast(const SelArgs& A, int sel, uint8_t* smem) {
  namespace cg = cooperative_groups;
  cg::cluster_group cl = cg::this_cluster();
  SelFastSmem& S = *reinterpret_cast<SelFastSmem*>(smem);
  uint32_t* sbits = reinterpret_cast<uint32_t*>(smem + sizeof(SelClusterSmem));  // this CTA's words
  const int tid = threadIdx.x, lane = tid & 31;
  const int r = (int)cl.block_rank();
  asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");  // every CTA started (before remote stores)
  const int B = A.B;
  const int per = B / kSelCL;
  const int wpc = per >> 5;
  const int k0 = r * per;
  uint8_t* rec = A.recs[sel];
  const uint64_t* keys = A.keys + (int64_t)sel * B;
  const uint4* h4 = reinterpret_cast<const uint4*>(A.hist0 + (int64_t)sel * 4096) + 4 * tid;  // bins [16 tid, 16 tid + 16)
  if (sel == 0 && r == 0) TRACE(10);
  constexpr int KC = 8;
  uint4 hb[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) hb[j] = __ldcg(h4 + j);
  uint64_t kb[KC];
#pragma unroll
  for (int u = 0; u < KC; ++u) {
    const int i = u * kSelCNT + tid;
    kb[u] = i < per ? __ldcg(keys + k0 + i) : 0ull;
  }
  if (tid == 0) S.lkey_n = 0;
  // 1. boundary digit: keys in bins above thread t's 16 = exclusive scan in reversed thread order
  uint32_t hv[16];
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    hv[4 * j] = hb[j].x; hv[4 * j + 1] = hb[j].y; hv[4 * j + 2] = hb[j].z; hv[4 * j + 3] = hb[j].w;
  }
  int mys = 0;
#pragma unroll
  for (int j = 0; j < 16; ++j) mys += (int)hv[j];
  int tot;
  // block_excl_scan over threads in descending order: thread t gets sum over t' > t
  {
    const int wid = tid >> 5;
    // reverse within the block: lane l of warp w plays position (255 - tid)
    int v = mys, inc = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {  // suffix scan inside the warp (lanes above)
      const int y = __shfl_down_sync(kFull, inc, o);
      if (lane + o < 32) inc += y;
    }
    if (lane == 0) S.sm[wid] = inc;  // warp total
    __syncthreads();
    int above_w = 0;
#pragma unroll
    for (int w = 0; w < kSelCNT / 32; ++w) above_w += w > wid ? S.sm[w] : 0;
    tot = 0;
#pragma unroll
    for (int w = 0; w < kSelCNT / 32; ++w) tot += S.sm[w];
    const int ex = above_w + inc - v;  // keys in bins of threads above me
    if (ex < A.num && A.num <= ex + mys) {
      int e = ex;
#pragma unroll
      for (int j = 15; j >= 0; --j) {
        const int c = (int)hv[j];
        if (e < A.num && A.num <= e + c) {
          S.pick[0] = 16 * tid + j;
          S.pick[1] = e;
          S.pick[2] = c;
        }
        e += c;
      }
    }
  }
  (void)tot;
  __syncthreads();
  const int d0 = S.pick[0];
  const int k2 = A.num - S.pick[1];
  const bool whole = (k2 == S.pick[2]);
  if (sel == 0 && r == 0) TRACE(11);
  // 2. classify my keys; candidates to my local list (fkey/fidx as scratch)
  const unsigned lt = (1u << lane) - 1u;
  int mytake = 0;
  for (int cb = 0; cb < per; cb += KC * kSelCNT) {
    if (cb > 0) {
#pragma unroll
      for (int u = 0; u < KC; ++u) {
        const int i = cb + u * kSelCNT + tid;
        kb[u] = i < per ? __ldcg(keys + k0 + i) : 0ull;
      }
    }
#pragma unroll
    for (int u = 0; u < KC; ++u) {
      const int i = cb + u * kSelCNT + tid;
      if (cb + u * kSelCNT >= per) break;
      const uint32_t d = (uint32_t)(kb[u] >> 51) & 0xFFFu;
      const bool take = i < per && (d > (uint32_t)d0 || (d == (uint32_t)d0 && whole));
      const bool cand = i < per && d == (uint32_t)d0 && !whole;
      const uint32_t word = __ballot_sync(kFull, take);
      if (lane == 0 && i < per) sbits[i >> 5] = word;  // per is a multiple of 32
      mytake += __popc(word);
      const unsigned cm = __ballot_sync(kFull, cand);
      if (cm) {
        int bpos = 0;
        if (lane == __ffs(cm) - 1) bpos = atomicAdd(&S.lkey_n, __popc(cm));
        bpos = __shfl_sync(kFull, bpos, __ffs(cm) - 1);
        if (cand) {
          const int pos = bpos + __popc(cm & lt);
          if (pos < kSelFastCap) {
            S.fkey[pos] = kb[u];
            S.fidx[pos] = k0 + i;
          }
        }
      }
    }
  }
  if (lane == 0) S.sm[8 + (tid >> 5)] = mytake;  // warp totals (every lane holds the warp's count)
  __syncthreads();
  const int nmine = S.lkey_n;
  asm volatile("barrier.cluster.wait.aligned;" ::: "memory");  // every CTA has started: remote stores allowed
  if (tid < kSelCL) {
    int t = 0;
#pragma unroll
    for (int w = 0; w < kSelCNT / 32; ++w) t += S.sm[8 + w];
    SelFastSmem* D = cl.map_shared_rank(&S, tid);
    D->take[r] = t;
    D->ncand[r] = nmine;
  }
  const int ncopy = min(nmine, kSelFastCap);
  for (int j = tid; j < ncopy * kSelCL; j += kSelCNT) {
    const int c = j / ncopy, q = j - c * ncopy;
    SelFastSmem* D = cl.map_shared_rank(&S, c);
    D->ckey[r][q] = S.fkey[q];
    D->cidx[r][q] = S.fidx[q];
  }
  cl.sync();
  if (sel == 0 && r == 0) TRACE(12);
  // 3. every candidate and every take count are here
  int nc = 0, offs[kSelCL];
  bool over = false;
#pragma unroll
  for (int c = 0; c < kSelCL; ++c) {
    offs[c] = nc;
    nc += S.ncand[c];
    over |= S.ncand[c] > kSelFastCap;
  }
  if (over) return false;
  if (tid < kSelCL) S.wins[tid] = 0;
  if (!whole) {
    for (int j = tid; j < nc; j += kSelCNT) {
      int c = 0, base = 0;
#pragma unroll
      for (int q = 1; q < kSelCL; ++q)
        if (j >= offs[q]) {
          c = q;
          base = offs[q];
        }
      S.fkey[j] = S.ckey[c][j - base];
      S.fidx[j] = S.cidx[c][j - base];
    }
    __syncthreads();
    const int lper = __ffs(per) - 1;  // per = B / kSelCL is a power of two
    for (int j = tid; j < nc; j += kSelCNT) {  // thread per candidate: rank = candidates preferred to it
      const uint64_t mk = S.fkey[j];
      const int mi = S.fidx[j];
      int rank = 0;
#pragma unroll 4
      for (int c = 0; c < nc; ++c) {
        const uint64_t kc = S.fkey[c];  // same address for every thread: broadcast
        rank += (kc > mk) | ((kc == mk) & (S.fidx[c] < mi));
      }
      if (rank < k2) {
        atomicAdd(&S.wins[mi >> lper], 1);
        if (mi >= k0 && mi < k0 + per) atomicOr(&sbits[(mi - k0) >> 5], 1u << (mi & 31));
      }
    }
  }
  __syncthreads();
  int jofs = 0, total = 0;
#pragma unroll
  for (int c = 0; c < kSelCL; ++c) {
    const int cc = S.take[c] + S.wins[c];
    jofs += c < r ? cc : 0;
    total += cc;
  }
  const int wpt = (wpc + kSelCNT - 1) / kSelCNT;
  int cnt = 0;
  for (int w = tid * wpt; w < min(wpc, (tid + 1) * wpt); ++w) cnt += __popc(sbits[w]);
  int mine;
  int pos = block_excl_scan<kSelCNT>(cnt, &mine, S.sm);
  if (sel == 0 && r == 0) TRACE(13);
  select_cluster_write(A, rec, sbits, sel, r, wpc, wpt, k0, pos + jofs, total);
  if (sel == 0 && r == 0) TRACE(14);
  return true;
}

// The cluster selection of location slot `sel` by the calling cluster of kSelCL
// CTAs x kSelCNT threads; smem: sizeof(SelClusterSmem) + B / kSelCL / 8 bytes.
// Reads keys and histograms through L2 (__ldcg): they may have been written by
// other CTAs of the cluster in the same kernel (k_slot), before a cluster barrier.
__device__ __forceinline__ void select_cluster_body(const SelArgs& A, int sel, uint8_t* smem) {
  namespace cg = cooperative_groups;
  cg::cluster_group cl = cg::this_cluster();
  if (!A.threshold_mode && select_cluster_fast(A, sel, smem)) return;
  SelClusterSmem& S = *reinterpret_cast<SelClusterSmem*>(smem);
  uint32_t* sbits = reinterpret_cast<uint32_t*>(smem + sizeof(SelClusterSmem));  // this CTA's words
  const int tid = threadIdx.x, lane = tid & 31;
  const int r = (int)cl.block_rank();
  // no remote shared memory may be touched before every CTA of the cluster has
  // started: arrive now, wait before the first DSMEM store (step 1)
  asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
  const int B = A.B;
  const int per = B / kSelCL;           // keys per CTA (multiple of 32)
  const int wpc = per >> 5;             // words per CTA
  const int k0 = r * per;
  uint8_t* rec = A.recs[sel];
  const uint64_t* keys = A.keys + (int64_t)sel * B;
  const uint32_t* h0 = A.hist0 + (int64_t)sel * 4096;
  if (sel == 0 && r == 0) TRACE(10);
#ifdef CUSFFT_TRACE
  const long long scs0 = clock64();
#define SELT(slot) CTRACE_MAX(slot, clock64() - scs0)
#else
#define SELT(slot) do { } while (0)
#endif
  // my keys (first chunk) and my two level-0 bins, all in flight at once
  constexpr int KC = 8;
  constexpr int BPC = 4096 / kSelCL;    // bins per CTA; thread t holds bins base, base - 1 (descending)
  const int hbase = r * BPC + BPC - 1 - 2 * tid;
  int c0 = 0, c1 = 0;
  if (!A.threshold_mode) {
    c0 = (int)__ldcg(h0 + hbase);
    c1 = (int)__ldcg(h0 + hbase - 1);
  }
  uint64_t kb[KC];
#pragma unroll
  for (int u = 0; u < KC; ++u) {
    const int i = u * kSelCNT + tid;
    kb[u] = i < per ? __ldcg(keys + k0 + i) : 0ull;
  }
  if (r == 0 && tid == 0) S.ncand = 0;
  int d0 = 0, k2 = 0;
  bool whole = true;
  {
  // 1. slice totals, pushed to every CTA of the cluster (once every CTA of the
  //    cluster has started: the split barrier's arrive was issued at entry)
  int tot, ex = 0;
  if (!A.threshold_mode) ex = block_excl_scan<kSelCNT>(c0 + c1, &tot, S.sm);
  SELT(117);
  asm volatile("barrier.cluster.wait.aligned;" ::: "memory");
  SELT(118);
  if (!A.threshold_mode && tid < kSelCL) cl.map_shared_rank(&S, tid)->part[r] = tot;
  cl.sync();
  SELT(119);
  // 2. the boundary slice (slices descending r = kSelCL-1 .. 0) finds d0 and pushes it
  if (!A.threshold_mode) {
    int above = 0, bs = 0;
#pragma unroll
    for (int c = kSelCL - 1; c >= 0; --c) {
      const int pc = S.part[c];
      if (above + pc >= A.num) { bs = c; break; }
      above += pc;
    }
    if (r == bs) {
      const int e = ex + above, kr = A.num;
      int pk0 = -1, pk1 = 0, pk2 = 0;
      if (e < kr && kr <= e + c0) { pk0 = hbase; pk1 = e; pk2 = c0; }
      else if (e + c0 < kr && kr <= e + c0 + c1) { pk0 = hbase - 1; pk1 = e + c0; pk2 = c1; }
      if (pk0 >= 0)
        for (int c = 0; c < kSelCL; ++c) {
          int* dst = cl.map_shared_rank(&S, c)->pick;
          dst[0] = pk0; dst[1] = pk1; dst[2] = pk2;
        }
    }
    cl.sync();
    SELT(120);
    d0 = S.pick[0];
    k2 = A.num - S.pick[1];
    whole = (k2 == S.pick[2]);
  }
  }
  if (sel == 0 && r == 0) TRACE(11);
  // 3. classify my keys: bitmap words in my smem, candidates appended to CTA 0,
  //    my count of keys taken outright pushed to every CTA
  SelClusterSmem* S0 = cl.map_shared_rank(&S, 0);
  const unsigned lt = (1u << lane) - 1u;
  if (tid == 0) S.sm[44] = 0;
  __syncthreads();
  for (int cb = 0; cb < per; cb += KC * kSelCNT) {
    if (cb > 0) {
#pragma unroll
      for (int u = 0; u < KC; ++u) {
        const int i = cb + u * kSelCNT + tid;
        kb[u] = i < per ? __ldcg(keys + k0 + i) : 0ull;
      }
    }
#pragma unroll
    for (int u = 0; u < KC; ++u) {
      const int i = cb + u * kSelCNT + tid;
      if (cb + u * kSelCNT >= per) break;
      const uint32_t d = (uint32_t)(kb[u] >> 51) & 0xFFFu;
      const bool take = i < per && (A.threshold_mode ? kb[u] >= A.thr_key : (d > (uint32_t)d0 || (d == (uint32_t)d0 && whole)));
      const bool cand = i < per && !A.threshold_mode && d == (uint32_t)d0 && !whole;
      const uint32_t word = __ballot_sync(kFull, take);
      if (lane == 0 && i < per) {  // per is a multiple of 32: whole warps in or out
        sbits[i >> 5] = word;
        atomicAdd(&S.sm[44], __popc(word));
      }
      const unsigned cm = __ballot_sync(kFull, cand);
      if (cm) {
        int bpos = 0;
        if (lane == __ffs(cm) - 1) bpos = atomicAdd(&S0->ncand, __popc(cm));
        bpos = __shfl_sync(kFull, bpos, __ffs(cm) - 1);
        if (cand) {
          const int pos = bpos + __popc(cm & lt);
          if (pos < kSelCap) {
            S0->ckey[pos] = kb[u];
            S0->cidx[pos] = k0 + i;
          }
        }
      }
    }
  }
  __syncthreads();
  SELT(121);
  if (tid < kSelCL) cl.map_shared_rank(&S, tid)->cnt[r] = S.sm[44];
  cl.sync();
  SELT(122);
  if (sel == 0 && r == 0) TRACE(12);
  // 4. the boundary bin's candidates.  Few (<= kSelCNT, the usual case): every
  //    CTA copies the whole list, ranks every candidate and so knows every
  //    CTA's final count (no further cluster round; CTA 0's list must outlive
  //    the copies: arrive on a split cluster barrier now, wait before exit).
  //    Many: every CTA resolves its own candidates, counts pushed in one more
  //    cluster round.
#ifdef CUSFFT_TRACE
  if (r == 0 && tid == 0 && sel < 16) g_trace[96 + sel] = (unsigned long long)S0->ncand | ((unsigned long long)whole << 32);
#endif
  const int nc = whole ? 0 : S0->ncand;
  const bool few = nc <= kSelCNT;
  int wins[kSelCL];
#pragma unroll
  for (int c = 0; c < kSelCL; ++c) wins[c] = 0;
  if (!whole) {
    Prefix96 p{0, 0, 0, 0};
    or96(p.phi, p.plo, (uint32_t)d0, pass_shift(0));
    or96(p.mhi, p.mlo, 0xFFFu, pass_shift(0));
    if (nc <= kSelCap) {
      if (r != 0)  // local copy of the candidate list (one remote round trip per thread)
        for (int c = tid; c < nc; c += kSelCNT) {
          S.ckey[c] = S0->ckey[c];
          S.cidx[c] = S0->cidx[c];
        }
      if (few) asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
      if (tid < kSelCL) S.part[tid] = 0;  // winners per CTA (reuses the slice totals)
      __syncthreads();
      SELT(123);
      if (few) {  // warp per candidate (every candidate), lanes split the comparisons
        for (int j = tid >> 5; j < nc; j += kSelCNT / 32) {
          const int mi = S.cidx[j];
          const int rank = warp_rank(S.ckey, S.cidx, nc, S.ckey[j], mi);
          if (lane == 0 && rank < k2) {
            atomicAdd(&S.part[mi / per], 1);
            if (mi >= k0 && mi < k0 + per) atomicOr(&sbits[(mi - k0) >> 5], 1u << (mi & 31));
          }
        }
      } else {
        p = block_radix_select<PairSrc, kSelCNT>(PairSrc{S.ckey, S.cidx}, nc, k2, S.hist, S.sm, 1, p, false);
        for (int c = tid; c < nc; c += kSelCNT) {
          const int mi = S.cidx[c];
          if (mi >= k0 && mi < k0 + per && ge96(p, S.ckey[c], ~(uint32_t)mi)) atomicOr(&sbits[(mi - k0) >> 5], 1u << (mi & 31));
        }
      }
    } else {  // crowded boundary bin: every CTA runs the radix over all keys of the bin, keeps its own
      p = block_radix_select<GKeySrc, kSelCNT>(GKeySrc{keys}, B, k2, S.hist, S.sm, 1, p, false);
      for (int i = tid; i < per; i += kSelCNT) {
        const uint64_t kk = __ldcg(keys + k0 + i);
        if (((kk >> 51) & 0xFFFu) == (uint32_t)d0 && ge96(p, kk, ~(uint32_t)(k0 + i)))
          atomicOr(&sbits[i >> 5], 1u << (i & 31));
      }
    }
    __syncthreads();
    SELT(124);
    if (few) {
#pragma unroll
      for (int c = 0; c < kSelCL; ++c) wins[c] = S.part[c];
    }
  }
  const int wpt = (wpc + kSelCNT - 1) / kSelCNT;
  int cnt = 0;
  for (int w = tid * wpt; w < min(wpc, (tid + 1) * wpt); ++w) cnt += __popc(sbits[w]);
  int mine;
  int pos = block_excl_scan<kSelCNT>(cnt, &mine, S.sm);
  SELT(125);
  if (!whole && !few) {  // resolved locally: my final count to every CTA
    if (tid < kSelCL) cl.map_shared_rank(&S, tid)->cnt[r] = mine;
    cl.sync();
  }
  if (sel == 0 && r == 0) TRACE(13);
  // 5. bitmap words and my part of the ascending J
  int jofs = 0, total = 0;
  const bool exact_counts = whole || few;  // S.cnt holds taken-outright counts; add the candidate winners
#pragma unroll
  for (int c = 0; c < kSelCL; ++c) {
    const int cc = S.cnt[c] + (exact_counts ? wins[c] : 0);
    jofs += c < r ? cc : 0;
    total += cc;
  }
  select_cluster_write(A, rec, sbits, sel, r, wpc, wpt, k0, pos + jofs, total);
  SELT(126);
#undef SELT
  if (sel == 0 && r == 0) TRACE(14);
  if (!whole && few && nc <= kSelCap) asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
  // (no remote smem access after the last barrier: CTAs may exit)
}

__global__ void __launch_bounds__(kSelCNT, 1) k_select_cluster(SelArgs A) {
  pdl_wait();
  KTRACE(8);
  extern __shared__ __align__(16) uint8_t smem[];
  select_cluster_body(A, blockIdx.x / kSelCL, smem);
}

// ---------------------------------------------------------------------------
// Step 3 (pass 2, L87) fused with Step 4 (L89, the exact cutoff) for the
// location slots: one cluster of kSelCL CTAs per location slot, CTA r owning
// rows k1 in [r ROWS, r ROWS + ROWS) of the four-step FFT (B = B1 x M, B1 =
// kSelCL ROWS).  Nothing of the cutoff goes through global memory:
//   1. the CTA loads its ROWS contiguous rows of v (pass 1's output), runs the
//      M-point row FFTs in shared memory and writes u^[k1 + B1 k2] to the
//      record; keys bits(|u^|^2) stay in shared memory and are counted into a
//      4096-bin top-digit histogram whose nonzero bins are added into every
//      CTA's copy (remote shared-memory atomics); cluster barrier;
//   2. every CTA finds the boundary digit d0 from the complete histogram,
//      classifies its keys and stores its ROWS-bit pieces of the slot's take
//      bitmap (bucket b = k1 + B1 k2: the piece of row k2 is bits [r ROWS,
//      r ROWS + ROWS) of the B1 buckets B1 k2 ...) into every CTA, and pushes
//      its boundary-bin candidates; cluster barrier;
//   3. every CTA holds the whole take bitmap and every candidate: it ranks
//      the candidates (ties to the smaller bucket), ORs the winners in, and
//      writes buckets [r B/kSelCL, (r+1) B/kSelCL) of the bitmap, the vote
//      table and the ascending J (offsets by one block scan of popcounts).
// Same u^ as k_fft, same winners and J as the cutoff kernels.  When a CTA
// holds more than kSelFastCap candidates the cluster falls back to the
// general cluster selection over the keys and histogram it also wrote to
// global memory.
// ---------------------------------------------------------------------------
struct Fft2SelArgs {
  SelArgs s;
  const double2* v[kMaxSel];  // pass-1 output of location slot i: row k1 = v[k1 M ... k1 M + M)
  const double2* tw;          // e^{-2 pi i t / B}, t < B
  int B1;
};

constexpr int kF2SNT = 1024;  // threads per CTA of k_fft2_select (32 warps: the chain is latency-bound)

template <int M, int ROWS>
__host__ __device__ constexpr int fft2sel_smem_bytes() {
  return fft_pad_n(M * ROWS) * 16 + M * 16 + 2 * 4096 * 4 + M * ROWS * 8 + M * ROWS * kSelCL / 8 +
         (int)sizeof(SelFastSmem) + kF2SNT * 4;
}

template <int M, int ROWS>
__global__ void __launch_bounds__(kF2SNT, 1) k_fft2_select(Fft2SelArgs F) {
  pdl_wait();
  KTRACE(8);
  namespace cg = cooperative_groups;
  cg::cluster_group cl = cg::this_cluster();
  constexpr int NT = kF2SNT;
  constexpr int E = M * ROWS;  // elements (and keys) of this CTA
  constexpr int EPT = E / NT;
  constexpr int HB = 4096 / NT;            // histogram bins per thread
  constexpr int WORDS = E * kSelCL / 32;   // bitmap words of the slot
  constexpr int WT = (WORDS + NT - 1) / NT;  // words per thread in the offset scan
  static_assert(E % NT == 0 && (ROWS == 8 || ROWS == 16 || ROWS == 32) && M <= NT, "fft2_select shape");
  const SelArgs& A = F.s;
  extern __shared__ __align__(16) uint8_t smem[];
  double2* S = reinterpret_cast<double2*>(smem);                 // fft_pad_n(E) (padded FFT workspace)
  double2* twl = S + fft_pad_n(E);                                // omega_M^t, t < M
  uint32_t* lh = reinterpret_cast<uint32_t*>(twl + M);           // 4096: my keys' top digits
  uint32_t* gh = lh + 4096;                                      // 4096: the slot's (summed over the cluster)
  uint64_t* skey = reinterpret_cast<uint64_t*>(gh + 4096);       // E: key of local t = k2 ROWS + j
  uint32_t* full = reinterpret_cast<uint32_t*>(skey + E);        // WORDS: the slot's bitmap
  SelFastSmem& C = *reinterpret_cast<SelFastSmem*>(full + WORDS);
  int* pre = reinterpret_cast<int*>(&C + 1);                     // NT: offset scan
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int r = (int)cl.block_rank();
  const int sel = blockIdx.x / kSelCL;
  const int B = A.B, B1 = F.B1;
  if (sel == 0 && r == 0) TRACE(10);
#ifdef CUSFFT_TRACE
  const long long fcs0 = clock64();
#define F2T(slot) CTRACE_MAX(slot, clock64() - fcs0)
#else
#define F2T(slot) do { } while (0)
#endif
  {
    const double2* vin = F.v[sel] + (int64_t)r * E;
    double2 buf[EPT];
#pragma unroll
    for (int u = 0; u < EPT; ++u) buf[u] = __ldcg(vin + u * NT + tid);
    // histograms zeroed before this CTA's arrive: the others add into gh only after their wait
#pragma unroll
    for (int j = 0; j < HB; ++j) {
      lh[j * NT + tid] = 0;
      gh[j * NT + tid] = 0;
    }
    if (tid == 0) C.lkey_n = 0;
    asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
    if (tid < M) twl[tid] = __ldg(F.tw + (int64_t)tid * (B / M));
#pragma unroll
    for (int u = 0; u < EPT; ++u) S[fft_pad(u * NT + tid)] = buf[u];
  }
  __syncthreads();
  F2T(117);
  fft_smem<M, E, NT, true>(S, twl, M);  // ROWS sequences of M: S[j M + k2] = row j's k2-th output
  F2T(118);
  uint8_t* rec = A.recs[sel];
  double2* uh = reinterpret_cast<double2*>(rec);
  uint64_t* gkeys = const_cast<uint64_t*>(A.keys) + (int64_t)sel * B;
#pragma unroll
  for (int u = 0; u < EPT; ++u) {
    const int t = u * NT + tid;
    const int j = t % ROWS, k2 = t / ROWS;
    const double2 val = S[fft_pad(j * M + k2)];
    const int b = r * ROWS + j + B1 * k2;
    uh[b] = val;
    const uint64_t key = (uint64_t)__double_as_longlong(__dadd_rn(__dmul_rn(val.x, val.x), __dmul_rn(val.y, val.y)));
    skey[t] = key;
    gkeys[b] = key;  // the general fallback reads keys and histogram through L2
    atomicAdd(&lh[(uint32_t)(key >> 51) & 0xFFFu], 1u);
  }
  __syncthreads();
  F2T(119);
  asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
  F2T(120);
#pragma unroll
  for (int j = 0; j < HB; ++j) {
    const int i = j * NT + tid;
    const uint32_t c = lh[i];
    if (c) {
      atomicAdd(A.hist0 + (int64_t)sel * 4096 + i, c);
#pragma unroll
      for (int q = 0; q < kSelCL; ++q) {
        const uint32_t ra = (uint32_t)__cvta_generic_to_shared(gh + i);
        uint32_t rq;
        asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(rq) : "r"(ra), "r"(q));
        asm volatile("red.shared::cluster.add.u32 [%0], %1;" ::"r"(rq), "r"(c) : "memory");
      }
    }
  }
  F2T(121);
  cl.sync();
  F2T(122);
  if (sel == 0 && r == 0) TRACE(11);
  // 2. boundary digit (every CTA alike): keys in the bins of higher threads by a reversed scan
  {
    uint32_t hv[HB];
    int mys = 0;
#pragma unroll
    for (int j = 0; j < HB; ++j) {
      hv[j] = gh[HB * tid + j];
      mys += (int)hv[j];
    }
    int inc = mys;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_down_sync(kFull, inc, o);
      if (lane + o < 32) inc += y;
    }
    if (lane == 0) C.sm[wid] = inc;
    __syncthreads();
    int above_w = 0;
    if (lane < NT / 32) above_w = lane > wid ? C.sm[lane] : 0;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) above_w += __shfl_xor_sync(kFull, above_w, o);
    const int ex = above_w + inc - mys;
    if (ex < A.num && A.num <= ex + mys) {
      int e = ex;
#pragma unroll
      for (int j = HB - 1; j >= 0; --j) {
        const int c = (int)hv[j];
        if (e < A.num && A.num <= e + c) {
          C.pick[0] = HB * tid + j;
          C.pick[1] = e;
          C.pick[2] = c;
        }
        e += c;
      }
    }
  }
  __syncthreads();
  const int d0 = C.pick[0];
  const int k2sel = A.num - C.pick[1];
  const bool whole = (k2sel == C.pick[2]);
  const unsigned lt = (1u << lane) - 1u;
#pragma unroll
  for (int u = 0; u < EPT; ++u) {
    const int t = u * NT + tid;
    const uint64_t key = skey[t];
    const uint32_t d = (uint32_t)(key >> 51) & 0xFFFu;
    const bool take = d > (uint32_t)d0 || (d == (uint32_t)d0 && whole);
    const bool cand = d == (uint32_t)d0 && !whole;
    const uint32_t word = __ballot_sync(kFull, take);
    // this warp's 32 keys = 32 / ROWS pieces (rows k2 = t0 / ROWS ...) of ROWS bits each
    const int t0 = t - lane;
    if (ROWS == 32) {
      if (lane < kSelCL) *cl.map_shared_rank(full + ((B1 * (t0 / ROWS) + r * ROWS) >> 5), lane) = word;
    } else if (ROWS == 16) {
      if (lane < 2 * kSelCL) {
        const int p = lane / kSelCL, q = lane % kSelCL;
        const int k2 = t0 / ROWS + p;
        uint16_t* dst = reinterpret_cast<uint16_t*>(full) + ((B1 * k2 + r * ROWS) >> 4);
        *cl.map_shared_rank(dst, q) = (uint16_t)(word >> (16 * p));
      }
    } else {
      const int p = lane / kSelCL, q = lane % kSelCL;  // 4 pieces x 8 CTAs
      const int k2 = t0 / ROWS + p;
      uint8_t* dst = reinterpret_cast<uint8_t*>(full) + ((B1 * k2 + r * ROWS) >> 3);
      *cl.map_shared_rank(dst, q) = (uint8_t)(word >> (8 * p));
    }
    const unsigned cm = __ballot_sync(kFull, cand);
    if (cm) {
      int bpos = 0;
      if (lane == __ffs(cm) - 1) bpos = atomicAdd(&C.lkey_n, __popc(cm));
      bpos = __shfl_sync(kFull, bpos, __ffs(cm) - 1);
      if (cand) {
        const int pos = bpos + __popc(cm & lt);
        if (pos < kSelFastCap) {
          C.fkey[pos] = key;
          C.fidx[pos] = r * ROWS + t % ROWS + B1 * (t / ROWS);
        }
      }
    }
  }
  __syncthreads();
  {
    const int nmine = C.lkey_n;
    if (tid < kSelCL) cl.map_shared_rank(&C, tid)->ncand[r] = nmine;
    const int ncopy = min(nmine, kSelFastCap);
    for (int j = tid; j < ncopy * kSelCL; j += NT) {
      const int q = j / ncopy, c = j - q * ncopy;
      SelFastSmem* D = cl.map_shared_rank(&C, q);
      D->ckey[r][c] = C.fkey[c];
      D->cidx[r][c] = C.fidx[c];
    }
  }
  F2T(123);
  cl.sync();
  F2T(124);
  if (sel == 0 && r == 0) TRACE(12);
  // 3. resolution, identical in every CTA
  int nc = 0, offs[kSelCL];
  bool over = false;
#pragma unroll
  for (int c = 0; c < kSelCL; ++c) {
    offs[c] = nc;
    nc += C.ncand[c];
    over |= C.ncand[c] > kSelFastCap;
  }
  if (over) {  // crowded boundary bin: CTA 0 runs the single-CTA selection over the keys and histogram in L2
    __threadfence();
    cl.sync();
    if (r == 0) select1_body(A, sel, smem, true);
    return;
  }
  if (!whole) {
    for (int j = tid; j < nc; j += NT) {
      int c = 0, base = 0;
#pragma unroll
      for (int q = 1; q < kSelCL; ++q)
        if (j >= offs[q]) {
          c = q;
          base = offs[q];
        }
      C.fkey[j] = C.ckey[c][j - base];
      C.fidx[j] = C.cidx[c][j - base];
    }
    __syncthreads();
    for (int j = tid; j < nc; j += NT) {
      const uint64_t mk = C.fkey[j];
      const int mi = C.fidx[j];
      int rank = 0;
#pragma unroll 4
      for (int c = 0; c < nc; ++c) {
        const uint64_t kc = C.fkey[c];
        rank += (kc > mk) | ((kc == mk) & (C.fidx[c] < mi));
      }
      if (rank < k2sel) atomicOr(&full[mi >> 5], 1u << (mi & 31));
    }
    __syncthreads();
  }
  // offsets: popcounts of the whole bitmap, WT words per thread
  int cnt = 0;
#pragma unroll
  for (int w = 0; w < WT; ++w) cnt += tid * WT + w < WORDS ? __popc(full[tid * WT + w]) : 0;
  int total;
  pre[tid] = block_excl_scan<NT>(cnt, &total, C.sm);
  __syncthreads();
  F2T(125);
  if (sel == 0 && r == 0) TRACE(13);
  const int wpc = WORDS / kSelCL;  // my words: [r wpc, r wpc + wpc), one per thread (wpc <= NT)
  int pos = 0;
  if (tid < wpc) {
    const int w = r * wpc + tid;
    pos = pre[w / WT];
    for (int q = (w / WT) * WT; q < w; ++q) pos += __popc(full[q]);
  }
  select_cluster_write<NT>(A, rec, full + r * wpc, sel, r, wpc, 1, r * E, pos, total);
  F2T(126);
#undef F2T
  if (sel == 0 && r == 0) TRACE(14);
}

// ---------------------------------------------------------------------------
// Step 4, Alg. 3 (L238-L250) as an ablation: one CTA of 1024 threads per
// location slot sorts all B (|u^|^2, bucket) pairs in shared memory (bitonic,
// larger key first, ties to the smaller bucket) and keeps the first num.
// Same winners as k_select; B <= 16384.  Dynamic smem: B x (u64 + int) + B/8.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(1024) k_select_sort(SelArgs A) {
  pdl_wait();
  KTRACE(8);
  extern __shared__ __align__(16) uint8_t smem[];
  const int B = A.B, tid = threadIdx.x;
  uint64_t* sk = reinterpret_cast<uint64_t*>(smem);
  int* si = reinterpret_cast<int*>(sk + B);
  uint32_t* sbits = reinterpret_cast<uint32_t*>(si + B);
  __shared__ int sm[40];
  const int sel = blockIdx.x;
  uint8_t* rec = A.recs[sel];
  const uint64_t* keys = A.keys + (int64_t)sel * B;
  const int words = (B + 31) >> 5;
  for (int i = tid; i < B; i += 1024) {
    sk[i] = __ldg(keys + i);
    si[i] = i;
  }
  for (int w = tid; w < words; w += 1024) sbits[w] = 0;
  __syncthreads();
  // "a before b" iff key_a > key_b or (key_a == key_b and idx_a < idx_b)
  for (int size = 2; size <= B; size <<= 1) {
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
      for (int t = tid; t < (B >> 1); t += 1024) {
        const int i = 2 * t - (t & (stride - 1));
        const int jn = i + stride;
        const bool up = (i & size) == 0;
        const uint64_t ka = sk[i], kb = sk[jn];
        const int ia = si[i], ib = si[jn];
        const bool b_first = (kb > ka) || (kb == ka && ib < ia);
        if (b_first == up) {
          sk[i] = kb;
          sk[jn] = ka;
          si[i] = ib;
          si[jn] = ia;
        }
      }
      __syncthreads();
    }
  }
  for (int r = tid; r < A.num; r += 1024) atomicOr(&sbits[si[r] >> 5], 1u << (si[r] & 31));
  __syncthreads();
  const SelOut so = sel_out(A, sel, rec);
  uint32_t* bitmap = so.bitmap;
  int* J = so.J;
  const int wpt = (words + 1023) >> 10;
  int cnt = 0;
  for (int w = tid * wpt; w < min(words, (tid + 1) * wpt); ++w) {
    bitmap[w] = sbits[w];
    cnt += __popc(sbits[w]);
  }
  int total;
  int pos = block_excl_scan<1024>(cnt, &total, sm);
  for (int w = tid * wpt; w < min(words, (tid + 1) * wpt); ++w) {
    uint32_t bits = sbits[w];
    while (bits) {
      const int b = __ffs(bits) - 1;
      bits &= bits - 1;
      J[pos++] = w * 32 + b;
    }
  }
  if (tid == 0) {
    *so.cnt = total;
    if (total != A.num) atomicOr(A.status + 1, 1);
  }
}

// ---------------------------------------------------------------------------
// Step 5 (L91-L93, Alg. 4).  bucket_q(f) = ((sigma_q f + nb/2) mod n) / nb
// is Alg. 4's range [ceil((J-1/2) nb), ceil((J+1/2) nb)).  A frequency with
// >= T of L_loc votes is selected in at least one of the first L_loc - T + 1
// location loops, so candidates f = a_{q0} p are enumerated only from those
// loops' preimage ranges, one warp per (q0, J) range, and f is counted at the
// first loop q0 that selects it: it needs T-1 votes among the later loops and
// none before q0.  The first min(L_loc-T-q0+1, later) later loops are probed
// branch-free (if all miss, f is rejected); the rare survivors probe the rest
// and then check the earlier loops.
// Dynamic smem: L_loc * ceil(B/32) u32 bitmaps.
// ---------------------------------------------------------------------------
constexpr int kMaxLoc = 32;  // location loops per plan (kernel-argument arrays)

struct VoteArgs {
  // per location loop, in vote order, by value (no dependent loads):
  const uint32_t* bmp[kMaxLoc];  // cutoff bitmap in the exchange buffer
  const int* Jp[kMaxLoc];        // ascending winner list
  const int* cntp[kMaxLoc];      // its length (num, or the Alg. 6 count)
  uint32_t sig[kMaxLoc];         // sigma
  uint32_t aa[kMaxLoc];          // a = sigma^-1
  const uint32_t* loc_sigma;     // the same sigmas in global memory (register-resident loads)
  int Lloc, T, num, B, nb, log2nb, log2n, log2B;
  int pairs;      // pair enumeration (T > ceil(L_loc / 2))
  int cnt_fixed;  // every winner list holds exactly num buckets (EXACT / SORT cutoffs)
  uint32_t nmask;
  int* hits;
  unsigned* hit_count;
  int max_hits;
  const uint32_t* pk;  // k_tail: the vote table already built by the cutoff (or null: transpose bmp)
};

// Scaled arithmetic: with F = f << (32 - log2 n), sigma * F + (nb/2 << (32 - log2 n))
// wraps at 2^32 exactly like (sigma f + nb/2) mod n scaled, so the bucket is
// the top log2 B bits: one IMAD + one shift, no mask.
__device__ __forceinline__ uint32_t lds_u32(uint32_t saddr) {
  uint32_t v;
  asm("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(saddr));
  return v;
}

// probe with a 32-bit shared address of loop q's bitmap
__device__ __forceinline__ uint32_t probe_sa(uint32_t row_s, uint32_t sig, uint32_t F, uint32_t half_s, int bsh) {
  const uint32_t h = sig * F + half_s;
  const uint32_t w = lds_u32(row_s + ((h >> (bsh + 5)) << 2));
  return __funnelshift_r(w, w, h >> bsh) & 1u;
}

// Survivors of the mandatory probes finish here, one per lane (convergent):
// the remaining later loops and the "no vote before q0" check.
__device__ __forceinline__ bool vote_finish(const VoteArgs& A, uint32_t bm_s, const uint32_t* ssig, int words,
                                            int q0, int m, uint32_t F, int got, uint32_t half_s, int bsh) {
  int votes = got;
  for (int q = q0 + 1 + m; q < A.Lloc; ++q)
    votes += probe_sa(bm_s + (uint32_t)(q * words) * 4u, ssig[q], F, half_s, bsh);
  bool hit = votes >= A.T - 1;
  for (int q = 0; q < q0; ++q) hit = hit && !probe_sa(bm_s + (uint32_t)(q * words) * 4u, ssig[q], F, half_s, bsh);
  return hit;
}

__device__ __forceinline__ void vote_emit(const VoteArgs& A, bool hit, uint32_t f) {
  const int lane = threadIdx.x & 31;
  const unsigned ball = __ballot_sync(kFull, hit);
  if (ball) {
    unsigned base = 0;
    const int leader = __ffs(ball) - 1;
    if (lane == leader) base = atomicAdd(A.hit_count, (unsigned)__popc(ball));
    base = __shfl_sync(kFull, base, leader);
    if (hit) {
      const unsigned slot = base + __popc(ball & ((1u << lane) - 1));
      if ((int)slot < A.max_hits) A.hits[slot] = (int)f;
    }
  }
}

// One (q0, J) preimage range per warp, VC candidates per lane per step.
// M = mandatory probes m = min(L_loc - T - q0 + 1, L_loc - 1 - q0) at compile
// time (M == 0: runtime count mrt): a candidate with m - g > L_loc - T - q0
// misses among them cannot reach T - 1 later votes and is dropped.  Survivors
// are queued in shared memory (qF: scaled f, qG: votes so far) and finished
// 32 at a time (convergent).
constexpr int kVCmax = 4;
constexpr int kVQ = 32 + 32 * kVCmax;  // per-warp survivor queue capacity

template <int M, int VC>
__device__ __forceinline__ void vote_unit(const VoteArgs& A, const uint32_t* __restrict__ bm, const uint32_t* ssig,
                                          int words, int q0, uint32_t Jv, uint32_t a, int mrt, uint32_t* qF,
                                          uint8_t* qG) {
  constexpr int MM = M > 0 ? M : 1;
  const int lane = threadIdx.x & 31;
  const int sh = 32 - A.log2n, bsh = 32 - A.log2B;
  const uint32_t half = (uint32_t)(A.nb >> 1);
  const uint32_t half_s = half << sh;
  const int m = M > 0 ? M : mrt;
  const int allowed = A.Lloc - A.T - q0;
  // 32-bit shared addresses of the probed bitmaps; sigma from global so that
  // it stays in registers
  const uint32_t bm_s = (uint32_t)__cvta_generic_to_shared(bm);
  uint32_t base[MM];
  uint32_t sg[MM];
#pragma unroll
  for (int qq = 0; qq < MM; ++qq) {
    base[qq] = bm_s + (uint32_t)((q0 + 1 + qq) * words) * 4u;
    sg[qq] = __ldg(A.loc_sigma + q0 + 1 + qq);
  }
  const int wsh = bsh + 5;
  const uint32_t p0 = Jv * (uint32_t)A.nb - half;
  uint32_t F0 = a * ((p0 + (uint32_t)lane) << sh);
  const uint32_t d32 = a * (32u << sh);
  const uint32_t dstep = a * ((32u * VC) << sh);
  const unsigned lt = (1u << lane) - 1;
  int qn = 0;  // queued survivors (warp-uniform)
  for (int t0 = 0; t0 < A.nb; t0 += 32 * VC, F0 += dstep) {
    uint32_t F[VC];
    int g[VC];
#pragma unroll
    for (int c = 0; c < VC; ++c) {
      F[c] = F0 + (uint32_t)c * d32;
      g[c] = 0;
    }
    if (M > 0) {
#pragma unroll
      for (int qq = 0; qq < MM; ++qq) {
#pragma unroll
        for (int c = 0; c < VC; ++c) {
          const uint32_t h = sg[qq] * F[c] + half_s;
          const uint32_t w = lds_u32(base[qq] + ((h >> wsh) << 2));
          g[c] += __funnelshift_r(w, w, h >> bsh) & 1u;
        }
      }
    } else {
      for (int qq = 0; qq < m; ++qq) {
        const uint32_t row = bm_s + (uint32_t)((q0 + 1 + qq) * words) * 4u;
#pragma unroll
        for (int c = 0; c < VC; ++c) g[c] += probe_sa(row, ssig[q0 + 1 + qq], F[c], half_s, bsh);
      }
    }
    unsigned bal[VC];
    unsigned any = 0u;
#pragma unroll
    for (int c = 0; c < VC; ++c) {
      const bool sv = (t0 + c * 32 + lane < A.nb) && (m - g[c]) <= allowed;
      bal[c] = __ballot_sync(kFull, sv);
      any |= bal[c];
    }
    if (any) {
#pragma unroll
      for (int c = 0; c < VC; ++c) {
        if (bal[c] & (1u << lane)) {
          const int pos = qn + __popc(bal[c] & lt);
          qF[pos] = F[c];
          qG[pos] = (uint8_t)g[c];
        }
        qn += __popc(bal[c]);
      }
      __syncwarp();
      while (qn >= 32) {  // finish 32 queued survivors, one per lane
        const uint32_t Fq = qF[qn - 32 + lane];
        const int gq = qG[qn - 32 + lane];
        __syncwarp();
        qn -= 32;
        const bool hit = vote_finish(A, bm_s, ssig, words, q0, m, Fq, gq, half_s, bsh);
        vote_emit(A, hit, Fq >> sh);
      }
    }
  }
  if (qn > 0) {
    const bool has = lane < qn;
    const uint32_t Fq = has ? qF[lane] : 0u;
    const int gq = has ? qG[lane] : 0;
    __syncwarp();
    const bool hit = has && vote_finish(A, bm_s, ssig, words, q0, m, Fq, gq, half_s, bsh);
    vote_emit(A, hit, Fq >> sh);
  }
}

__global__ void __launch_bounds__(256) k_vote(VoteArgs A) {
  pdl_wait();
  KTRACE(9);
  extern __shared__ __align__(16) uint8_t smem[];
  if (blockIdx.x == 0) TRACE(30);
  uint32_t* bm = reinterpret_cast<uint32_t*>(smem);
  __shared__ uint32_t ssig[64];
  __shared__ uint32_t queueF[8][kVQ];
  __shared__ uint8_t queueG[8][kVQ];
  const int words = (A.B + 31) >> 5;
  if ((words & 3) == 0) {  // 16-B vector loads, all loops' words in flight before the first store
    const int lv4 = A.log2B - 7;  // log2(words / 4)
    const int tot = A.Lloc << lv4;
    constexpr int PER = 8;
    uint4* dst = reinterpret_cast<uint4*>(bm);
    for (int i0 = 0; i0 < tot; i0 += PER * (int)blockDim.x) {
      uint4 tmp[PER];
#pragma unroll
      for (int u = 0; u < PER; ++u) {
        const int i = i0 + u * blockDim.x + threadIdx.x;
        if (i < tot) tmp[u] = __ldg(reinterpret_cast<const uint4*>(A.bmp[i >> lv4]) + (i & ((1 << lv4) - 1)));
      }
#pragma unroll
      for (int u = 0; u < PER; ++u) {
        const int i = i0 + u * blockDim.x + threadIdx.x;
        if (i < tot) dst[i] = tmp[u];
      }
    }
  } else {
    for (int q = 0; q < A.Lloc; ++q)
      for (int i = threadIdx.x; i < words; i += blockDim.x) bm[q * words + i] = A.bmp[q][i];
  }
  __shared__ int scnt[kMaxLoc + 1];  // prefix sums of the enumerated loops' counts
  if (threadIdx.x < A.Lloc) ssig[threadIdx.x] = A.sig[threadIdx.x];
  if (threadIdx.x == 0) {
    int acc = 0;
    scnt[0] = 0;
    for (int q = 0; q <= A.Lloc - A.T; ++q) {
      acc += __ldg(A.cntp[q]);
      scnt[q + 1] = acc;
    }
  }
  __syncthreads();
  if (blockIdx.x == 0) TRACE(31);
  const int units = scnt[A.Lloc - A.T + 1];
  uint32_t* qF = queueF[threadIdx.x >> 5];
  uint8_t* qG = queueG[threadIdx.x >> 5];
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nwarps = (gridDim.x * blockDim.x) >> 5;
  for (int unit = warp; unit < units; unit += nwarps) {
    int q0 = 0;
    while (unit >= scnt[q0 + 1]) ++q0;
    const int jidx = unit - scnt[q0];
    const uint32_t Jv = (uint32_t)__ldg(A.Jp[q0] + jidx);
    const uint32_t a = A.aa[q0];
    const int m = min(A.Lloc - A.T - q0 + 1, A.Lloc - 1 - q0);  // mandatory probes
    switch (m) {
      case 1: vote_unit<1, 2>(A, bm, ssig, words, q0, Jv, a, 1, qF, qG); break;
      case 2: vote_unit<2, 2>(A, bm, ssig, words, q0, Jv, a, 2, qF, qG); break;
      case 3: vote_unit<3, 2>(A, bm, ssig, words, q0, Jv, a, 3, qF, qG); break;
      case 4: vote_unit<4, 2>(A, bm, ssig, words, q0, Jv, a, 4, qF, qG); break;
      default: vote_unit<0, 2>(A, bm, ssig, words, q0, Jv, a, m, qF, qG); break;
    }
  }
  TRACE_END(32);
}

// ---------------------------------------------------------------------------
// Step 6 (L95, Alg. 5), one warp per hit, one lane per loop (slot).
// For hit f and loop l:  p = sigma_l f mod n, h = p / nb, d = p mod nb;
//   if d > nb/2: h = h+1 mod B, d -= nb;
//   v_l = u^_l[h] * e^{-2 pi i tau_l f / n} / G^(-d);
// val = (element of rank (L-1)/2 of Re v) + i (same of Im v), ties by loop.
// Also counts the top digits of the output keys |val|^2 for k_output.
// ---------------------------------------------------------------------------
struct EstArgs {
  const uint8_t* records;
  RecLayout lay;
  const SlotParam* slots;
  int L;
  const double2* ginv;      // 1 / G^(q) of the location loops' filter, q = -nb/2 .. nb/2 (plan time)
  const double2* ginv_est;  // the same for loops r >= ghat_split (the estimation-only filter)
  int ghat_split;           // L_loc with separate filters, else L
  const double2* ph_hi;     // e^{-2 pi i (j << plo) / n}, j < n >> plo   (plan time)
  const double2* ph_lo;     // e^{-2 pi i j / n}, j < 2^plo
  int plo;
  const int* hits;
  const unsigned* hit_count;
  int max_hits;
  uint32_t nmask;
  int log2nb, nb, B;
  double n;
  double2* hit_vals;
  uint64_t* hit_keys;
  double2* per_loop;  // may be null
  uint32_t* out_hist;  // [4096] level-0 histogram of hit_keys
};


// v_l = u^_l[h] e^{-2 pi i tau_l f / n} / G^(-d) (Alg. 5 L311-L325 with the
// permutation's phase removed [Z4]).  The phase e^{-2 pi i m / n}, m = tau f
// mod n, is the product of two plan-time table entries (m's high and low
// bits, each computed by sincospi of an exact fraction) and the division by
// G^ a multiplication by its plan-time reciprocal: every load of the
// estimate is independent, so its latency is one L2 round trip.
__device__ __forceinline__ double2 loop_estimate(const EstArgs& A, const SlotParam& sp, int l, uint32_t f) {
  const uint32_t p = (sp.sigma * f) & A.nmask;
  int hb = (int)(p >> A.log2nb);
  int d = (int)(p & (uint32_t)(A.nb - 1));
  if (d > (A.nb >> 1)) {
    hb = (hb + 1) & (A.B - 1);
    d -= A.nb;
  }
  const uint32_t tph = (sp.tau * f) & A.nmask;
  const double2 gi = __ldg((sp.loop < (uint32_t)A.ghat_split ? A.ginv : A.ginv_est) + (A.nb >> 1) - d);  // 1 / G^(-d)
  const double2 b = __ldg(reinterpret_cast<const double2*>(A.records + (int64_t)l * A.lay.rec_bytes) + hb);
  const double2 e1 = __ldg(A.ph_hi + (tph >> A.plo));
  const double2 e0 = __ldg(A.ph_lo + (tph & ((1u << A.plo) - 1u)));
  const double2 ph = make_double2(e1.x * e0.x - e1.y * e0.y, e1.x * e0.y + e1.y * e0.x);
  const double zr = b.x * ph.x - b.y * ph.y;  // b * e^{-i phi}
  const double zi = b.x * ph.y + b.y * ph.x;
  return make_double2(zr * gi.x - zi * gi.y, zr * gi.y + zi * gi.x);
}

// Element of rank `med` among the L values held as (lane: a0 = slot lane,
// a1 = slot lane + 32); ties ordered by slot.  Returns it on every lane.
__device__ __forceinline__ double warp_rank_select(double a0, double a1, int L, int med) {
  const int lane = threadIdx.x & 31;
  int r0 = 0, r1 = 0;
  const int L0 = min(L, 32);
  for (int j = 0; j < L0; ++j) {
    const double v = __shfl_sync(kFull, a0, j);
    r0 += (v < a0) || (v == a0 && j < lane);
    r1 += (v < a1) || (v == a1);  // slot j < 32 <= slot of a1
  }
  for (int j = 32; j < L; ++j) {
    const double v = __shfl_sync(kFull, a1, j - 32);
    r0 += (v < a0);
    r1 += (v < a1) || (v == a1 && j < lane + 32);
  }
  const bool h0 = lane < L0 && r0 == med;
  const bool h1 = lane + 32 < L && r1 == med;
  const unsigned b = __ballot_sync(kFull, h0 || h1);
  const int src = __ffs(b) - 1;
  const double mine = h0 ? a0 : a1;
  return __shfl_sync(kFull, mine, src);
}

__global__ void __launch_bounds__(256) k_estimate(EstArgs A) {
  pdl_launch_dependents();
  pdl_wait();
  KTRACE(10);
  __shared__ uint32_t sdig[8];
  if (blockIdx.x == 0) TRACE(40);
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  SlotParam sp0{0, 0, 0, 0}, sp1{0, 0, 0, 0};
  if (lane < A.L) sp0 = A.slots[lane];
  if (lane + 32 < A.L) sp1 = A.slots[lane + 32];
  const int H = min((int)*A.hit_count, A.max_hits);
  const int med = (A.L - 1) >> 1;
  for (int h0 = blockIdx.x * 8; h0 < H; h0 += gridDim.x * 8) {  // CTA-uniform
    const int h = h0 + wib;
    uint32_t dig = 0xFFFFFFFFu;
    if (h < H) {
      const uint32_t f = (uint32_t)__ldg(A.hits + h);
      double2 v0 = make_double2(0.0, 0.0), v1 = make_double2(0.0, 0.0);
      if (lane < A.L) v0 = loop_estimate(A, sp0, lane, f);
      if (lane + 32 < A.L) v1 = loop_estimate(A, sp1, lane + 32, f);
      if (A.per_loop) {
        if (lane < A.L) A.per_loop[(int64_t)h * A.L + lane] = v0;
        if (lane + 32 < A.L) A.per_loop[(int64_t)h * A.L + lane + 32] = v1;
      }
      const double vr = warp_rank_select(v0.x, v1.x, A.L, med);
      const double vi = warp_rank_select(v0.y, v1.y, A.L, med);
      const uint64_t key = (uint64_t)__double_as_longlong(__dadd_rn(__dmul_rn(vr, vr), __dmul_rn(vi, vi)));
      if (lane == 0) {
        A.hit_vals[h] = make_double2(vr, vi);
        A.hit_keys[h] = key;
      }
      dig = (uint32_t)(key >> 51) & 0xFFFu;
    }
    if (lane == 0) sdig[wib] = dig;
    __syncthreads();
    if (threadIdx.x < 8) {  // one atomic per distinct digit of this CTA's 8 hits
      const uint32_t d = sdig[threadIdx.x];
      bool first = d != 0xFFFFFFFFu;
      uint32_t c = 0;
      for (int j = 0; j < 8; ++j) {
        first = first && !(j < (int)threadIdx.x && sdig[j] == d);
        c += sdig[j] == d;
      }
      if (first) atomicAdd(A.out_hist + d, c);
    }
    __syncthreads();
  }
  TRACE_END(41);
}

// Segmented form for L <= LP (LP = 8 or 16): a warp holds 32 / LP hits, one
// segment of LP lanes per hit, lane li of a segment = loop li; the same
// per-loop estimate and the same rank rule (ties by loop) inside the segment.
// Twice (L = 16) the hits per warp of k_estimate with all 32 lanes busy.
template <int LP>
__global__ void __launch_bounds__(256) k_estimate_seg(EstArgs A) {
  pdl_launch_dependents();
  pdl_wait();
  KTRACE(10);
  constexpr int G = 32 / LP;    // hits per warp
  constexpr int NH = 8 * G;     // hits per CTA iteration
  __shared__ uint32_t sdig[NH];
  if (blockIdx.x == 0) TRACE(40);
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int seg = lane / LP, li = lane % LP, sbase = seg * LP;
  const bool act = li < A.L;
  SlotParam sp{0, 0, 0, 0};
  if (act) sp = A.slots[li];
  const int H = min((int)*A.hit_count, A.max_hits);
  const int med = (A.L - 1) >> 1;
  const unsigned segmask = (LP == 32 ? kFull : ((1u << LP) - 1u)) << sbase;
  for (int h0 = blockIdx.x * NH; h0 < H; h0 += gridDim.x * NH) {  // CTA-uniform
    const int h = h0 + wib * G + seg;
    const bool valid = h < H;
    double2 v = make_double2(0.0, 0.0);
    if (valid && act) {
      const uint32_t f = (uint32_t)__ldg(A.hits + h);
      v = loop_estimate(A, sp, li, f);
      if (A.per_loop) A.per_loop[(int64_t)h * A.L + li] = v;
    }
    // element of rank med among the segment's L values (ties by loop), re and im separately
    double vr = 0.0, vi = 0.0;
#pragma unroll
    for (int part = 0; part < 2; ++part) {
      const double a = part ? v.y : v.x;
      int r = 0;
#pragma unroll
      for (int j = 0; j < LP; ++j) {
        const double b = __shfl_sync(kFull, a, sbase + j);
        r += (j < A.L) && ((b < a) || (b == a && j < li));
      }
      const unsigned bal = __ballot_sync(kFull, act && r == med) & segmask;
      const int src = bal ? __ffs(bal) - 1 : sbase;
      const double m = __shfl_sync(kFull, a, src);
      if (part) vi = m; else vr = m;
    }
    uint32_t dig = 0xFFFFFFFFu;
    if (valid) {
      const uint64_t key = (uint64_t)__double_as_longlong(__dadd_rn(__dmul_rn(vr, vr), __dmul_rn(vi, vi)));
      if (li == 0) {
        A.hit_vals[h] = make_double2(vr, vi);
        A.hit_keys[h] = key;
      }
      dig = (uint32_t)(key >> 51) & 0xFFFu;
    }
    if (li == 0) sdig[wib * G + seg] = dig;
    __syncthreads();
    if (threadIdx.x < NH) {  // one atomic per distinct digit of this CTA's hits
      const uint32_t d = sdig[threadIdx.x];
      bool first = d != 0xFFFFFFFFu;
      uint32_t c = 0;
      for (int j = 0; j < NH; ++j) {
        first = first && !(j < (int)threadIdx.x && sdig[j] == d);
        c += sdig[j] == d;
      }
      if (first) atomicAdd(A.out_hist + d, c);
    }
    __syncthreads();
  }
  TRACE_END(41);
}

}  // namespace cusfft
