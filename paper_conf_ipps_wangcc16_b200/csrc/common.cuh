// common.cuh — shared device primitives of the CUDA path (block scans, the
// 96-bit radix select used by the cutoff and the output selection).
// Product code only: nothing here is shared with oracle/.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace cusfft {

constexpr unsigned kFull = 0xFFFFFFFFu;

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

// Block-wide radix select (blockDim.x == 1024): find a prefix such that the
// items with ge96(prefix, item) are exactly the K largest composites among N.
// src.get(i, hi, lo) must be callable for 0 <= i < N.  Requires 1 <= K <= N.
// hist: 4096 u32 in shared memory; sm: >= 40 ints in shared memory.
// Digits: 12 bits MSB-first; bit 95 (the sign of a non-negative fp64 key) is
// skipped; early exit once the boundary digit's whole bin is selected.
template <class Src>
__device__ Prefix96 block_radix_select(const Src& src, int N, int K, uint32_t* hist, int* sm) {
  constexpr int NT = 1024;
  const int tid = threadIdx.x, lane = tid & 31;
  Prefix96 p{0, 0, 0, 0};
  int krem = K;
  for (int pass = 0; pass < 8; ++pass) {
    const int shift = pass < 7 ? 83 - 12 * pass : 0;
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
    // thread t owns bins 4095-4t .. 4092-4t (descending digit order)
    const int base = 4095 - 4 * tid;
    const int c0 = hist[base], c1 = hist[base - 1], c2 = hist[base - 2], c3 = hist[base - 3];
    const int mine = c0 + c1 + c2 + c3;
    int total;
    const int ex = block_excl_scan<NT>(mine, &total, sm);
    if (ex < krem && krem <= ex + mine) {
      int cum = ex, d, cnt;
      if (cum + c0 >= krem) {
        d = base; cnt = c0;
      } else if ((cum += c0) + c1 >= krem) {
        d = base - 1; cnt = c1;
      } else if ((cum += c1) + c2 >= krem) {
        d = base - 2; cnt = c2;
      } else {
        cum += c2; d = base - 3; cnt = c3;
      }
      sm[32] = d; sm[33] = cum; sm[34] = cnt;
    }
    __syncthreads();
    const uint32_t d = (uint32_t)sm[32];
    const int above = sm[33], cnt = sm[34];
    __syncthreads();
    or96(p.phi, p.plo, d, shift);
    or96(p.mhi, p.mlo, 0xFFFu, shift);
    krem -= above;
    if (cnt == krem) break;  // every item in the boundary bin is selected
  }
  return p;
}

}  // namespace cusfft
