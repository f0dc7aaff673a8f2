// exchange.cuh — the two-collective loop-sharded finish (shard_mode 2,
// SURVEY.md §8(e) steps 1-5; BASELINE north_star: "candidate-index and
// per-loop estimate lists combined by NCCL allgather"):
//
//   local   Steps 1-4 of this rank's loops; the cutoff writes its location
//           loops' candidate records (bitmap | count | ascending J) into
//           this rank's slice of the candidate buffer
//   #1      all-gather of the candidate buffer (L_loc records)
//   mid     every rank votes over all location loops (identical hit SET,
//           PAPER.md:L91-L93, Alg. 4), sorts the hits ascending
//           (the appends are unordered; the sort makes the hit list, and so
//           the per-loop estimate slices, identical on every rank), and
//           estimates ITS loops for every hit (Alg. 5)
//   #2      all-gather of the per-loop estimates [rank][hit][local loop]
//   finish  median over all L loops per hit, re and im separately (L95,
//           Alg. 5), then the output selection (k_output)
//
// Per-loop estimates come from the same loop_estimate as the fused tail, so
// the result is bit-identical to a single-GPU plan.
#pragma once
#include "tail.cuh"

namespace cusfft {

// Ascending sort of the hit list in place (one CTA of 1024 threads, bitonic
// over the next power of two >= H in shared memory; smem: npow2(max_hits) x 4
// bytes).  Hits are distinct frequencies, so the order is unique.
constexpr int kSortNT = 1024;
__global__ void __launch_bounds__(kSortNT) k_hits_sort(int* __restrict__ hits, const unsigned* __restrict__ hit_count,
                                                       int max_hits) {
  pdl_wait();
  extern __shared__ __align__(16) int shv[];
  const int H = min((int)*hit_count, max_hits);
  int N = 2;
  while (N < H) N <<= 1;
  for (int i = threadIdx.x; i < N; i += kSortNT) shv[i] = i < H ? __ldcg(hits + i) : 0x7fffffff;
  __syncthreads();
  for (int size = 2; size <= N; size <<= 1) {
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
      for (int t = threadIdx.x; t < (N >> 1); t += kSortNT) {
        const int i = 2 * t - (t & (stride - 1));
        const int j = i + stride;
        const bool up = (i & size) == 0;
        const int a = shv[i], b = shv[j];
        if ((a > b) == up) {
          shv[i] = b;
          shv[j] = a;
        }
      }
      __syncthreads();
    }
  }
  for (int i = threadIdx.x; i < H; i += kSortNT) hits[i] = shv[i];
}

// This rank's per-loop estimates v_s(f) for every hit f (slots slot0 ..
// slot0 + Lg - 1 of the records, which this rank computed): x2[h][i] for
// local slot i.  Thread per (hit, local slot).
__global__ void __launch_bounds__(256) k_est_local(EstArgs E, int slot0, int Lg, double2* __restrict__ x2) {
  pdl_wait();
  const int H = min((int)*E.hit_count, E.max_hits);
  const int total = H * Lg;
  for (int idx = blockIdx.x * blockDim.x + threadIdx.x; idx < total; idx += gridDim.x * blockDim.x) {
    const int h = idx / Lg, i = idx - h * Lg;
    const SlotParam sp = E.slots[slot0 + i];
    x2[idx] = loop_estimate(E, sp, slot0 + i, (uint32_t)__ldcg(E.hits + h));
  }
}

// Median of the L = G x Lg per-loop estimates of hit h (x2: [G][max_hits][Lg]
// after the all-gather; rank g's local slot i is slot g Lg + i), element of
// rank floor((L-1)/2) of the real and of the imaginary parts, ties by slot
// (as the fused tail).  Writes the hit value, its key |val|^2 and the output
// histogram; debug plans also the per-loop values in slot order.
constexpr int kMedMaxL = 64;
__global__ void __launch_bounds__(128) k_median(EstArgs E, const double2* __restrict__ x2, int G, int Lg) {
  pdl_wait();
  const int H = min((int)*E.hit_count, E.max_hits);
  const int L = G * Lg;
  const int med = (L - 1) >> 1;
  for (int h = blockIdx.x * blockDim.x + threadIdx.x; h < H; h += gridDim.x * blockDim.x) {
    double re[kMedMaxL], im[kMedMaxL];
    for (int g = 0; g < G; ++g)
      for (int i = 0; i < Lg; ++i) {
        const double2 v = __ldcg(x2 + ((int64_t)g * E.max_hits + h) * Lg + i);
        re[g * Lg + i] = v.x;
        im[g * Lg + i] = v.y;
        if (E.per_loop) E.per_loop[(int64_t)h * L + g * Lg + i] = v;
      }
    double vr = 0.0, vi = 0.0;
    for (int s = 0; s < L; ++s) {
      int rr = 0, ri = 0;
      for (int j = 0; j < L; ++j) {
        rr += (re[j] < re[s]) || (re[j] == re[s] && j < s);
        ri += (im[j] < im[s]) || (im[j] == im[s] && j < s);
      }
      if (rr == med) vr = re[s];
      if (ri == med) vi = im[s];
    }
    const uint64_t key = (uint64_t)__double_as_longlong(__dadd_rn(__dmul_rn(vr, vr), __dmul_rn(vi, vi)));
    E.hit_vals[h] = make_double2(vr, vi);
    E.hit_keys[h] = key;
    atomicAdd(E.out_hist + ((uint32_t)(key >> 51) & 0xFFFu), 1u);
  }
}

}  // namespace cusfft
