// common.cuh — shared device primitives of the CUDA path (block scans, the
// 96-bit radix select used by the cutoff and the output selection).
// Product code only: nothing here is shared with oracle/.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace cusfft {

constexpr unsigned kFull = 0xFFFFFFFFu;

// Opt-in phase tracing (build with -DCUSFFT_TRACE): TRACE(slot) stores the
// %globaltimer (ns) of thread 0 of the calling CTA into g_trace[slot].
#ifdef CUSFFT_TRACE
__device__ unsigned long long g_trace[256];
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define TRACE(slot) \
  do { if (threadIdx.x == 0) g_trace[(slot)] = gtimer(); } while (0)
#define TRACE_END(slot) \
  do { if (threadIdx.x == 0) atomicMax(&g_trace[(slot)], gtimer()); } while (0)
// Per-kernel span: g_trace[128 + 2 id] = earliest CTA start (after pdl_wait),
// g_trace[129 + 2 id] = latest CTA end (thread 0; any return path).
// Per-CTA records (start, end, id | smid << 8 | linear block << 16) in g_cta.
constexpr int kCtaTraceMax = 16384;
__device__ unsigned g_cta_n;
__device__ unsigned long long g_cta[3 * kCtaTraceMax];
struct KTraceScope {
  int id;
  unsigned long long t0;
  __device__ explicit KTraceScope(int i) : id(i), t0(0) {
    if (threadIdx.x == 0) {
      t0 = gtimer();
      atomicMin(&g_trace[128 + 2 * id], t0);
    }
  }
  __device__ ~KTraceScope() {
    if (threadIdx.x == 0) {
      const unsigned long long t1 = gtimer();
      atomicMax(&g_trace[129 + 2 * id], t1);
      unsigned smid;
      asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
      const unsigned i = atomicAdd(&g_cta_n, 1u);
      if (i < kCtaTraceMax) {
        g_cta[3 * i] = t0;
        g_cta[3 * i + 1] = t1;
        g_cta[3 * i + 2] = (unsigned long long)id | ((unsigned long long)smid << 8) |
                           ((unsigned long long)(blockIdx.x + blockIdx.y * gridDim.x) << 16);
      }
    }
  }
};
#define KTRACE(id) KTraceScope ktrace_scope_(id)
// SM-clock stamps (cheap to read; differences only within one CTA):
// CTRACE(slot) stores clock64() of thread 0; CTRACE_MAX(slot, cycles) keeps the largest value.
#define CTRACE(slot) \
  do { if (threadIdx.x == 0) g_trace[(slot)] = (unsigned long long)clock64(); } while (0)
#define CTRACE_MAX(slot, v) \
  do { if (threadIdx.x == 0) atomicMax(&g_trace[(slot)], (unsigned long long)(v)); } while (0)
#else
#define CTRACE(slot) do { } while (0)
#define CTRACE_MAX(slot, v) do { } while (0)
#define KTRACE(id) do { } while (0)
#define TRACE(slot) do { } while (0)
#define TRACE_END(slot) do { } while (0)
#endif

// Programmatic dependent launch: a kernel launched with programmatic stream
// serialization may start while its predecessor drains; it must not touch
// global memory the predecessor writes (or reads) before this wait.  No-op
// for ordinary launches.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

// Early launch of the dependent kernel (programmatic dependent launch): its
// CTAs become resident and block in pdl_wait until this grid completes.
// Used where measured faster (the fallback chain's estimation -> output;
// early-resident successors elsewhere slowed their predecessors).
__device__ __forceinline__ void pdl_launch_dependents() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

// Bulk (TMA engine) global -> shared copies completing on an mbarrier.
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
// bytes: multiple of 16; both addresses 16-B aligned.  L2 policy: evict-first.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra WAIT_%=;\n}" ::"r"(
          smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// Per-slot loop parameters (slot order; see DESIGN.md §6 "slots").
//   sigma: gather stride (Alg. 1's ai), a = sigma^-1 mod n,
//   tau: offset (Def. 1), loop: the loop index r this slot holds.
struct SlotParam {
  uint32_t sigma, tau, a, loop;
};

__device__ __forceinline__ int warp_incl_scan(int v) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int t = __shfl_up_sync(kFull, v, o);
    if (lane >= o) v += t;
  }
  return v;
}

// Exclusive block scan for blockDim.x == NT (multiple of 32, <= 1024).
// sm must hold >= 32 ints.  Returns the exclusive prefix; *total = block sum.
template <int NT>
__device__ __forceinline__ int block_excl_scan(int v, int* total, int* sm) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int inc = warp_incl_scan(v);
  if (lane == 31) sm[wid] = inc;
  __syncthreads();
  if (wid == 0) {
    int w = (lane < NT / 32) ? sm[lane] : 0;
    int wi = warp_incl_scan(w);
    sm[lane] = wi;
  }
  __syncthreads();
  int off = wid ? sm[wid - 1] : 0;
  *total = sm[NT / 32 - 1];
  __syncthreads();
  return off + inc - v;
}

// ---------------------------------------------------------------------------
// 96-bit composite keys: (hi = 64-bit key, lo = ~index).  Larger composite is
// preferred: larger key first, then smaller index (the tie rule of the cutoff
// and of the output selection, DESIGN.md §3 [Z9]).  All composites of one
// selection are distinct, so "the K largest" is a unique set.
// ---------------------------------------------------------------------------
struct Prefix96 {
  uint64_t phi, mhi;
  uint32_t plo, mlo;
};

__device__ __forceinline__ uint32_t digit96(uint64_t hi, uint32_t lo, int shift) {
  if (shift >= 32) return (uint32_t)(hi >> (shift - 32)) & 0xFFFu;
  return (uint32_t)(((hi << (32 - shift)) | (uint64_t)(lo >> shift)) & 0xFFFull);
}

__device__ __forceinline__ void or96(uint64_t& hi, uint32_t& lo, uint32_t d, int shift) {
  if (shift >= 32) {
    hi |= (uint64_t)d << (shift - 32);
  } else {
    lo |= d << shift;
    if (shift > 20) hi |= (uint64_t)(d >> (32 - shift));
  }
}

__device__ __forceinline__ bool match96(const Prefix96& p, uint64_t hi, uint32_t lo) {
  return ((hi & p.mhi) == p.phi) && ((lo & p.mlo) == p.plo);
}

// masked(composite) >= prefix, lexicographic over 96 bits.
__device__ __forceinline__ bool ge96(const Prefix96& p, uint64_t hi, uint32_t lo) {
  uint64_t h = hi & p.mhi;
  if (h != p.phi) return h > p.phi;
  return (lo & p.mlo) >= p.plo;
}

// Digit shift of radix pass `pass` (12-bit digits MSB-first; bit 95, the sign
// of a non-negative fp64 key, is skipped; the last pass overlaps one bit).
__device__ __forceinline__ int pass_shift(int pass) { return pass < 7 ? 83 - 12 * pass : 0; }

// Block-wide scan of a 4096-bin histogram from the top digit down
// (blockDim.x == NT): returns {digit, count above it, count in it} of the
// bin holding the krem-th largest item.  Requires 1 <= krem <= total.
struct BinPick {
  int d, above, cnt;
};

template <int NT = 1024>
__device__ __forceinline__ BinPick pick_bin(const uint32_t* hist, int krem, int* sm) {
  constexpr int PER = 4096 / NT;  // bins per thread, descending
  const int tid = threadIdx.x;
  const int base = 4095 - PER * tid;
  int c[PER];
  int mine = 0;
#pragma unroll
  for (int j = 0; j < PER; ++j) {
    c[j] = hist[base - j];
    mine += c[j];
  }
  int total;
  const int ex = block_excl_scan<NT>(mine, &total, sm);
  if (ex < krem && krem <= ex + mine) {
    int cum = ex;
#pragma unroll
    for (int j = 0; j < PER; ++j) {
      if (cum + c[j] >= krem) {
        sm[32] = base - j; sm[33] = cum; sm[34] = c[j];
        break;
      }
      cum += c[j];
    }
  }
  __syncthreads();
  BinPick r{sm[32], sm[33], sm[34]};
  __syncthreads();
  return r;
}

// Block-wide radix select (blockDim.x == NT): find a prefix such that the
// items with ge96(prefix, item) are exactly the K largest composites among N.
// src.get(i, hi, lo) must be callable for 0 <= i < N.  Starts at radix pass
// `start` with the digits of earlier passes already fixed in `p` and `krem`
// items still to choose among those matching p (start = 0: p empty, krem = K).
// If `prebuilt`, hist already holds the counts of pass `start` (over the items
// matching p).  hist: 4096 u32 in shared memory; sm: >= 40 ints.
// Early exit once the boundary digit's whole bin is selected.
template <class Src, int NT = 1024>
__device__ Prefix96 block_radix_select(const Src& src, int N, int krem, uint32_t* hist, int* sm, int start = 0,
                                       Prefix96 p = Prefix96{0, 0, 0, 0}, bool prebuilt = false) {
  const int tid = threadIdx.x, lane = tid & 31;
  for (int pass = start; pass < 8; ++pass) {
    const int shift = pass_shift(pass);
    if (!(prebuilt && pass == start)) {
      for (int i = tid; i < 4096; i += NT) hist[i] = 0;
      __syncthreads();
      for (int i0 = 0; i0 < N; i0 += NT) {
        const int i = i0 + tid;
        bool valid = i < N;
        uint32_t d = 0xFFFFFFFFu;
        if (valid) {
          uint64_t hi;
          uint32_t lo;
          src.get(i, hi, lo);
          valid = match96(p, hi, lo);
          if (valid) d = digit96(hi, lo, shift);
        }
        const unsigned grp = __match_any_sync(kFull, d);
        if (valid && lane == __ffs(grp) - 1) atomicAdd(&hist[d], (uint32_t)__popc(grp));
      }
      __syncthreads();
    }
    const BinPick b = pick_bin<NT>(hist, krem, sm);
    or96(p.phi, p.plo, (uint32_t)b.d, shift);
    or96(p.mhi, p.mlo, 0xFFFu, shift);
    krem -= b.above;
    if (b.cnt == krem) break;  // every item in the boundary bin is selected
  }
  return p;
}

}  // namespace cusfft
