// exchange.cuh — the two-collective loop-sharded finish (shard_mode 2,
// SURVEY.md §8(e) steps 1-5; BASELINE north_star: "candidate-index and
// per-loop estimate lists combined by NCCL allgather"):
//
//   local   Steps 1-4 of this rank's loops; the cutoff writes its location
//           loops' candidate records (bitmap | count | ascending J) into
//           this rank's slice of the candidate buffer
//   #1      all-gather of the candidate buffer (L_loc records)
//   mid     every rank votes over all location loops (identical hit SET,
//           PAPER.md:L91-L93, Alg. 4; k_vote), ranks the hits
//           (the appends are unordered; ascending order makes the hit list,
//           and so the per-loop estimate slices, identical on every rank) and
//           estimates ITS loops for every hit (Alg. 5; k_rank_est)
//   #2      all-gather of the per-loop estimates [rank][hit][local loop]
//   finish  median over all L loops per hit, re and im separately (L95,
//           Alg. 5), then the output selection (k_output)
//
// Per-loop estimates come from the same loop_estimate as the fused tail, so
// the result is bit-identical to a single-GPU plan.
#pragma once
#include "tail.cuh"

namespace cusfft {

// The hit list in ascending order plus this rank's per-loop estimates, in one
// kernel: a CTA takes a chunk of kRankC hits of the (unordered) list from the
// vote; its warps count, over the whole list staged in shared memory
// (max_hits x 4 bytes), the hits smaller than each of them (hits are distinct frequencies, so the ranks are a
// permutation and the order is unique), the chunk's hits go to
// hits_sorted[rank], and the CTA estimates them for this rank's slots s =
// slot0 .. slot0 + Lg - 1 (the records this rank computed) into x2[rank][i].
constexpr int kRankNT = 256, kRankC = 32;
__global__ void __launch_bounds__(kRankNT) k_rank_est(EstArgs E, int slot0, int Lg, int* __restrict__ hits_sorted,
                                                      double2* __restrict__ x2) {
  pdl_wait();
  extern __shared__ __align__(16) int shl[];  // the whole hit list (max_hits entries)
  __shared__ int srank[kRankC];
  __shared__ uint32_t sf[kRankC];
  const int H = min((int)*E.hit_count, E.max_hits);
  const int h0 = blockIdx.x * kRankC;
  if (h0 >= H) return;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  for (int i = tid; i < H; i += kRankNT) shl[i] = __ldcg(E.hits + i);  // independent loads: one L2 round trip
  if (tid < kRankC) srank[tid] = 0;
  __syncthreads();
  // warp w counts, for every hit of the chunk (lane = chunk position), the
  // smaller hits among list entries j = w, w + 8, ... (broadcast reads)
  const int f = h0 + lane < H ? shl[h0 + lane] : 0;
  int r = 0;
#pragma unroll 8
  for (int j = wid; j < H; j += kRankNT / 32) r += shl[j] < f;
  atomicAdd(&srank[lane], r);
  if (tid < kRankC) sf[tid] = (uint32_t)(h0 + tid < H ? shl[h0 + tid] : 0);
  __syncthreads();
  const int nh = min(kRankC, H - h0);
  if (tid < nh) hits_sorted[srank[tid]] = (int)sf[tid];
  for (int w = tid; w < nh * Lg; w += kRankNT) {
    const int t = w / Lg, i = w - t * Lg;
    const SlotParam sp = E.slots[slot0 + i];
    x2[(int64_t)srank[t] * Lg + i] = loop_estimate(E, sp, slot0 + i, sf[t]);
  }
}

// Median of the L = G x Lg per-loop estimates of hit h (x2: [G][max_hits][Lg]
// after the all-gather; rank g's local slot i is slot g Lg + i): one warp per
// hit, lane l holding slots l and l + 32, the element of rank floor((L-1)/2)
// of the real and of the imaginary parts, ties by slot (warp_rank_select, as
// the fused tail).  Writes the hit value, its key |val|^2 and the output
// histogram; debug plans also the per-loop values in slot order.
constexpr int kMedMaxL = 64;  // two values per lane
__global__ void __launch_bounds__(256) k_median(EstArgs E, const double2* __restrict__ x2, int G, int Lg) {
  pdl_wait();
  const int H = min((int)*E.hit_count, E.max_hits);
  const int L = G * Lg;
  const int med = (L - 1) >> 1;
  const int lane = threadIdx.x & 31;
  const int nw = (gridDim.x * blockDim.x) >> 5;
  for (int h = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; h < H; h += nw) {  // warp-uniform
    double2 v0 = make_double2(0.0, 0.0), v1 = make_double2(0.0, 0.0);
    if (lane < L) v0 = __ldcg(x2 + ((int64_t)(lane / Lg) * E.max_hits + h) * Lg + lane % Lg);
    if (lane + 32 < L) v1 = __ldcg(x2 + ((int64_t)((lane + 32) / Lg) * E.max_hits + h) * Lg + (lane + 32) % Lg);
    if (E.per_loop) {
      if (lane < L) E.per_loop[(int64_t)h * L + lane] = v0;
      if (lane + 32 < L) E.per_loop[(int64_t)h * L + lane + 32] = v1;
    }
    const double vr = warp_rank_select(v0.x, v1.x, L, med);
    const double vi = warp_rank_select(v0.y, v1.y, L, med);
    if (lane == 0) {
      const uint64_t key = (uint64_t)__double_as_longlong(__dadd_rn(__dmul_rn(vr, vr), __dmul_rn(vi, vi)));
      E.hit_vals[h] = make_double2(vr, vi);
      E.hit_keys[h] = key;
      atomicAdd(E.out_hist + ((uint32_t)(key >> 51) & 0xFFFu), 1u);
    }
  }
}

}  // namespace cusfft
