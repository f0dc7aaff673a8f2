// tail.cuh — Steps 5 + 6 + output in ONE kernel (k_tail), after the cutoff:
//
//   Step 5  reverse hash + vote      PAPER.md:L91-L93, Alg. 4
//   Step 6  median estimation        PAPER.md:L95, Alg. 5
//   output  k strongest, by f        PAPER.md:L13 (k large coefficients), Alg. 5
//
// One CTA of 1024 threads per SM.  Every CTA holds the location loops' cutoff
// results as one table element per bucket (bit q = bucket kept in location
// loop q; uint8_t for L_loc <= 8, uint16_t <= 16, uint32_t <= 32) in shared
// memory, copied from the array the cluster cutoff ORs its winners into or
// transposed from the per-loop bitmaps.
//
// Vote (the candidate set is Alg. 4's: frequency f = a_q p for p in the
// preimage range [J n/B - n/(2B), J n/B + n/(2B)) of a kept bucket J of loop
// q, and f is a hit iff >= T location loops keep the bucket f hashes to; the
// GPU enumerates each hit exactly once instead of counting in a score[n]
// array):
//   * pairs (T > ceil(L_loc/2)): a hit has some pair (2i, 2i+1) voting twice,
//     so candidates run over loop 2i's ranges with ONE mandatory probe of loop
//     2i+1 (f counted at its first such pair);
//   * otherwise: candidates of loop q0 = 0 .. L_loc - T (f counted at its
//     first voting loop) with the probes of the next m loops as the filter.
// A warp owns one (enumerated loop, J) unit.  The mandatory probe of a
// candidate is IADD + SHF + LDS + LOP on a running scaled position: with
// F = f << (32 - log2 n) (exact mod-n arithmetic by 2^32 wrap-around), the
// probed loop's bucket is (sigma_q a_e (p << sh) + (n/2B << sh)) >> (32 - log2 B)
// and consecutive p add a constant.  A lane collects 32 candidates' survival
// bits in a mask; survivors are compacted through a per-warp queue and
// finished 32 at a time (probe every location loop, apply the rule).
//
// Estimation (fused): a warp estimates the hits its finish round produced,
// a 16-lane segment per hit (L <= 16; a whole warp per hit otherwise), lane
// = slot: p = sigma f mod n, bucket h, offset d (Alg. 5, d > n/2B
// moves to the next bucket), v = u^[h] e^{-2 pi i tau f/n} / G^(-d), and the
// element of rank floor((L-1)/2) of the real and of the imaginary parts (L95,
// Alg. 5; ties by slot).
//
// Output (fused): the last CTA to finish (threadfence + counter) selects the
// k hits of largest |val|^2 (ties to the smaller f) and writes them sorted by
// f (output_body, shared with the stand-alone k_output).
#pragma once
#include "exec_kernels.cuh"

namespace cusfft {

struct TailArgs {
  VoteArgs v;          // location loops in vote order: bitmaps, winner lists, sigma, a (pk: ET table or null)
  EstArgs e;           // every slot: records, slot params, G^, hit buffers, output-key histogram
  int k, kp2, log2n;
  int64_t* locs;
  double2* vals;
  int* status;         // d_flags + 1
  unsigned* done;      // finished-CTA counter (per-execution zero block)
  int q_off;           // byte offset of the per-warp queues in dynamic smem
};

constexpr int kTailNT = 1024;
constexpr int kTailQ = 1024;  // per-warp queue entries (u16 candidate offsets): one whole chunk

// Output selection (Alg. 5 L333-L335 emits all hits, the k
// strongest are kept [Z12]): the k hits of largest |val|^2 (ties to the
// smaller f), written in ascending f; pads loc = -1, val = 0.  blockDim.x ==
// 1024.  Two-level selection (level 0 counted by the estimation into ghist),
// then a bucket sort by the top 10 bits of f with a per-bucket insertion sort
// (bitonic fallback for crowded buckets).  smem: 4096 u32 hist + 64 ints +
// kOutCap x (u64 + int) + kp2 x u64 x 2 + 1024 x 2 ints.
constexpr int kOutCap = 4096;

// Dynamic smem of output_body: the layout above, then a 4096-bin copy of the
// level-0 histogram.
__host__ __device__ constexpr int output_smem_bytes(int kp2) {
  return 4096 * 4 + 64 * 4 + kOutCap * 12 + 2 * kp2 * 8 + 2 * 1024 * 4;
}
__host__ __device__ constexpr int output_smem_total(int kp2) { return output_smem_bytes(kp2) + 4096 * 4; }

__device__ void output_body(uint8_t* smem, const int* __restrict__ hits, const unsigned* hit_count, int max_hits,
                            const double2* __restrict__ hit_vals, const uint64_t* __restrict__ hit_keys,
                            uint32_t* __restrict__ ghist, int k, int kp2, int log2n, int64_t* __restrict__ locs,
                            double2* __restrict__ vals, int* __restrict__ status) {
  uint32_t* hist = reinterpret_cast<uint32_t*>(smem);
  int* sm = reinterpret_cast<int*>(smem + 4096 * 4);
  uint64_t* ckey = reinterpret_cast<uint64_t*>(smem + 4096 * 4 + 64 * 4);
  int* cidx = reinterpret_cast<int*>(ckey + kOutCap);
  uint64_t* sel = reinterpret_cast<uint64_t*>(cidx + kOutCap);  // (f << 32 | i), kp2 entries
  uint64_t* srt = sel + kp2;                                     // bucket-sorted copy
  int* bcnt = reinterpret_cast<int*>(srt + kp2);                 // 1024 bucket counters
  int* bstart = bcnt + 1024;                                     // 1024 bucket starts
  const int tid = threadIdx.x;
  TRACE(50);
  // the level-0 histogram through L2 into shared memory (other CTAs of k_tail
  // counted into it; it is the selection's read-only level 0 from here on)
  uint32_t* h0 = reinterpret_cast<uint32_t*>(smem + output_smem_bytes(kp2));
  for (int i = tid; i < 4096; i += 1024) h0[i] = __ldcg(ghist + i);
  ghist = h0;
  __syncthreads();
  const unsigned hc = __ldcg(hit_count);
  const int H = min((int)hc, max_hits);
  if (tid == 0 && (int)hc > max_hits) atomicOr(status, 1);
  const int K = min(k, H);
  // Fast path (H <= 16384 items, k <= 2048): every item's key, f and value
  // are loaded into registers while the level-0 boundary bin is found; if that
  // bin is taken whole (the usual case: the k planted coefficients stand far
  // above the false hits), one classification pass selects, and the values go
  // to shared memory (aliasing the unused candidate arrays).
  constexpr int PF = 4, NCH = 4;  // items per thread per chunk, chunks
  double2* selv = reinterpret_cast<double2*>(ckey);  // [kp2] values of the selected entries (fast path)
  const bool fast = H <= NCH * PF * 1024 && kp2 * 16 <= kOutCap * 12;
  uint64_t pk[PF];
  uint32_t pf[PF];
  double2 pv[PF];
  if (fast) {  // chunk 0: keys, f and values
#pragma unroll
    for (int u = 0; u < PF; ++u) {
      const int i = u * 1024 + tid;
      if (i < H) {
        pk[u] = __ldcg(hit_keys + i);
        pf[u] = (uint32_t)__ldcg(hits + i);
        pv[u] = __ldcg(hit_vals + i);
      }
    }
  }
  if (tid == 0) sm[41] = 0;
  bcnt[tid] = 0;
  bool direct = false;  // selv holds the values
  if (fast) {
    uint32_t d0 = 0;
    bool whole = true;
    if (H > K) {
      const BinPick b0 = pick_bin(ghist, K, sm);  // syncs
      d0 = (uint32_t)b0.d;
      whole = (K - b0.above) == b0.cnt;
    } else {
      __syncthreads();
    }
    if (whole) {
      direct = true;
      const int lane = tid & 31;
      for (int ch = 0; ch < NCH && ch * PF * 1024 < H; ++ch) {  // block-uniform
        if (ch > 0) {  // later chunks (many false hits): keys and f here, values only for the selected
#pragma unroll
          for (int u = 0; u < PF; ++u) {
            const int i = ch * PF * 1024 + u * 1024 + tid;
            if (i < H) {
              pk[u] = __ldcg(hit_keys + i);
              pf[u] = (uint32_t)__ldcg(hits + i);
            }
          }
        }
#pragma unroll
        for (int u = 0; u < PF; ++u) {
          const int i = ch * PF * 1024 + u * 1024 + tid;
          const bool take = i < H && ((uint32_t)(pk[u] >> 51) & 0xFFFu) >= d0;
          const unsigned bal = __ballot_sync(kFull, take);
          int base = 0;
          if (lane == 0 && bal) base = atomicAdd(&sm[41], __popc(bal));
          base = __shfl_sync(kFull, base, 0);
          if (take) {
            const int pos = base + __popc(bal & ((1u << lane) - 1u));
            if (pos < kp2) {
              sel[pos] = ((uint64_t)pf[u] << 32) | (uint32_t)pos;
              selv[pos] = ch == 0 ? pv[u] : __ldcg(hit_vals + i);
            }
          }
        }
      }
      __syncthreads();
    }
  } else {
    __syncthreads();
  }
  if (!direct) {
    auto add = [&](int i) {
      const int pos = atomicAdd(&sm[41], 1);
      if (pos < kp2) sel[pos] = ((uint64_t)(uint32_t)__ldcg(hits + i) << 32) | (uint32_t)i;
    };
    if (H > K) {
      select_topk(
          H, K, ghist,
          [&](int i, uint64_t& kk, uint32_t& t) {
            kk = __ldcg(hit_keys + i);
            t = (uint32_t)__ldcg(hits + i);
          },
          add, ckey, cidx, kOutCap, hist, sm);
    } else {
      for (int i = tid; i < H; i += 1024) add(i);
      __syncthreads();
    }
  }
  TRACE(51);
  const int ns = min(sm[41], kp2);
  if (tid == 0 && sm[41] != K) atomicOr(status + 2, 1);
  // bucket sort by the top 10 bits of f
  const int sh = max(0, log2n - 10);
  for (int i = tid; i < ns; i += 1024) atomicAdd(&bcnt[(int)(sel[i] >> 32) >> sh], 1);
  __syncthreads();
  const int c = bcnt[tid];
  int total;
  const int st = block_excl_scan<1024>(c, &total, sm);
  bstart[tid] = st;
  if (tid == 0) sm[42] = 0;
  __syncthreads();
  atomicMax(&sm[42], c);
  bcnt[tid] = 0;
  __syncthreads();
  for (int i = tid; i < ns; i += 1024) {
    const int bkt = (int)(sel[i] >> 32) >> sh;
    srt[bstart[bkt] + atomicAdd(&bcnt[bkt], 1)] = sel[i];
  }
  __syncthreads();
  if (sm[42] <= 32) {
    const int b0 = bstart[tid];
    for (int i = 1; i < c; ++i) {  // insertion sort of this thread's bucket
      const uint64_t v = srt[b0 + i];
      int j = i - 1;
      while (j >= 0 && srt[b0 + j] > v) {
        srt[b0 + j + 1] = srt[b0 + j];
        --j;
      }
      srt[b0 + j + 1] = v;
    }
  } else {  // crowded bucket: bitonic over all selected entries
    for (int i = ns + tid; i < kp2; i += 1024) srt[i] = ~0ull;
    __syncthreads();
    for (int size = 2; size <= kp2; size <<= 1) {
      for (int stride = size >> 1; stride > 0; stride >>= 1) {
        for (int t = tid; t < (kp2 >> 1); t += 1024) {
          const int i = 2 * t - (t & (stride - 1));
          const int jn = i + stride;
          const bool up = (i & size) == 0;
          const uint64_t a = srt[i], b = srt[jn];
          if ((a > b) == up) {
            srt[i] = b;
            srt[jn] = a;
          }
        }
        __syncthreads();
      }
    }
  }
  __syncthreads();
  TRACE(52);
  for (int j = tid; j < k; j += 1024) {
    if (j < ns) {
      const uint64_t v = srt[j];
      locs[j] = (int64_t)(v >> 32);
      vals[j] = direct ? selv[(uint32_t)v] : __ldcg(hit_vals + (uint32_t)v);
    } else {
      locs[j] = -1;
      vals[j] = make_double2(0.0, 0.0);
    }
  }
  TRACE(53);
}

// Stand-alone output kernel (the fallback chain: k_vote / k_estimate* / k_output).
__global__ void __launch_bounds__(1024) k_output(const int* __restrict__ hits, const unsigned* __restrict__ hit_count,
                                                 int max_hits, const double2* __restrict__ hit_vals,
                                                 const uint64_t* __restrict__ hit_keys, uint32_t* __restrict__ ghist,
                                                 int k, int kp2, int log2n, int64_t* __restrict__ locs,
                                                 double2* __restrict__ vals, int* __restrict__ status) {
  pdl_wait();
  KTRACE(11);
  extern __shared__ __align__(16) uint8_t smem[];
  output_body(smem, hits, hit_count, max_hits, hit_vals, hit_keys, ghist, k, kp2, log2n, locs, vals, status);
}


// Estimate the hits of one finish round (hit: this lane's candidate is a hit,
// f its frequency).  Warp-uniform control flow; all 32 lanes call it.
// LP = 16: a 16-lane segment per hit, lane li = slot li (L <= 16);
// LP = 32: a warp per hit, lanes hold slots li and li + 32 (L <= 64).
template <int LP>
__device__ __forceinline__ void tail_emit_estimate(const TailArgs& A, bool hit, uint32_t f, const SlotParam& sp0,
                                                   const SlotParam& sp1) {
  const int lane = threadIdx.x & 31;
  unsigned hb = __ballot_sync(kFull, hit);
  if (!hb) return;
  unsigned base = 0;
  const int leader = __ffs(hb) - 1;
  if (lane == leader) base = atomicAdd(A.v.hit_count, (unsigned)__popc(hb));
  base = __shfl_sync(kFull, base, leader);
  const unsigned myslot = base + __popc(hb & ((1u << lane) - 1u));
  if (hit && (int)myslot < A.v.max_hits) A.v.hits[myslot] = (int)f;
  const EstArgs& E = A.e;
  const int L = E.L;
  const int med = (L - 1) >> 1;
  constexpr int G = 32 / LP;  // hits per step
  while (hb) {  // warp-uniform
    int src[G];
#pragma unroll
    for (int g = 0; g < G; ++g) {
      src[g] = hb ? __ffs(hb) - 1 : -1;
      if (hb) hb &= hb - 1;
    }
    const int seg = lane / LP, li = lane % LP;
    int s = src[0];
#pragma unroll
    for (int g = 1; g < G; ++g)
      if (seg == g) s = src[g];
    const uint32_t hf = __shfl_sync(kFull, f, s < 0 ? 0 : s);
    const unsigned hs = __shfl_sync(kFull, myslot, s < 0 ? 0 : s);
    const bool valid = s >= 0 && (int)hs < A.v.max_hits;
    double vr, vi;
    if (LP == 16) {
      const unsigned segmask = 0xFFFFu << (seg * 16);
      const bool act = li < L;
      double2 v = make_double2(0.0, 0.0);
      if (valid && act) {
        v = loop_estimate(E, sp0, li, hf);
        if (E.per_loop) E.per_loop[(int64_t)hs * L + li] = v;
      }
#pragma unroll
      for (int part = 0; part < 2; ++part) {
        const double a = part ? v.y : v.x;
        int r = 0;
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          const double b = __shfl_sync(kFull, a, seg * 16 + j);
          r += (j < L) && ((b < a) || (b == a && j < li));
        }
        const unsigned bal = __ballot_sync(kFull, act && r == med) & segmask;
        const int from = bal ? __ffs(bal) - 1 : seg * 16;
        const double m = __shfl_sync(kFull, a, from);
        if (part) vi = m; else vr = m;
      }
    } else {
      double2 v0 = make_double2(0.0, 0.0), v1 = make_double2(0.0, 0.0);
      if (valid) {
        if (lane < L) v0 = loop_estimate(E, sp0, lane, hf);
        if (lane + 32 < L) v1 = loop_estimate(E, sp1, lane + 32, hf);
        if (E.per_loop) {
          if (lane < L) E.per_loop[(int64_t)hs * L + lane] = v0;
          if (lane + 32 < L) E.per_loop[(int64_t)hs * L + lane + 32] = v1;
        }
      }
      vr = warp_rank_select(v0.x, v1.x, L, med);
      vi = warp_rank_select(v0.y, v1.y, L, med);
    }
    if (valid && li == 0) {
      const uint64_t key = (uint64_t)__double_as_longlong(__dadd_rn(__dmul_rn(vr, vr), __dmul_rn(vi, vi)));
      E.hit_vals[hs] = make_double2(vr, vi);
      E.hit_keys[hs] = key;
      atomicAdd(E.out_hist + ((uint32_t)(key >> 51) & 0xFFFu), 1u);
    }
  }
}

template <typename ET>
__device__ __forceinline__ uint32_t tab_at(uint32_t base, uint32_t i) {
  uint32_t v;
  if (sizeof(ET) == 1)
    asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(base + i));
  else if (sizeof(ET) == 2)
    asm volatile("ld.shared.u16 %0, [%1];" : "=r"(v) : "r"(base + 2u * i));
  else
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(base + 4u * i));
  return v;
}

// ET: vote table element; LP: estimation lanes per hit (16 or 32).
template <typename ET, int LP>
__global__ void __launch_bounds__(kTailNT, 1) k_tail(TailArgs A) {
  pdl_wait();
  KTRACE(9);
  extern __shared__ __align__(16) uint8_t smem[];
  __shared__ uint32_t ssig[kMaxLoc], saa[kMaxLoc];
  __shared__ int scnt[kMaxLoc + 1];
  __shared__ int s_last;
  const VoteArgs& V = A.v;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  if (blockIdx.x == 0) TRACE(30);
  const int B = V.B, Lloc = V.Lloc;
  // ---- the vote table: copy (the cutoff ORed the winners into V.pk) or transpose the bitmaps
  if (V.pk) {
    const int n16 = (int)(((int64_t)B * sizeof(ET) + 15) / 16);
    for (int i = tid; i < n16; i += kTailNT)
      reinterpret_cast<uint4*>(smem)[i] = __ldcg(reinterpret_cast<const uint4*>(V.pk) + i);
  } else {
    ET* tab = reinterpret_cast<ET*>(smem);
    const int words = (B + 31) >> 5;
    for (int w = tid; w < words; w += kTailNT) {
      uint32_t bw[kMaxLoc];
#pragma unroll
      for (int q = 0; q < (int)(8 * sizeof(ET)); ++q) bw[q] = q < Lloc ? __ldcg(V.bmp[q] + w) : 0u;
      const int ne = min(32, B - 32 * w);
      for (int e = 0; e < ne; ++e) {
        uint32_t v = 0u;
#pragma unroll
        for (int q = 0; q < (int)(8 * sizeof(ET)); ++q) v |= ((bw[q] >> e) & 1u) << q;
        tab[32 * w + e] = (ET)v;
      }
    }
  }
  const int nenum = V.pairs ? Lloc / 2 : Lloc - V.T + 1;
  if (tid < Lloc) {
    ssig[tid] = V.sig[tid];
    saa[tid] = V.aa[tid];
  }
  if (tid == 0) {
    int acc = 0;
    scnt[0] = 0;
    for (int e = 0; e < nenum; ++e) {
      acc += __ldcg(V.cntp[V.pairs ? 2 * e : e]);
      scnt[e + 1] = acc;
    }
  }
  // slot parameters of the lanes' estimation slots
  SlotParam sp0{0, 0, 0, 0}, sp1{0, 0, 0, 0};
  {
    const int li = LP == 16 ? (lane & 15) : lane;
    if (li < A.e.L) sp0 = A.e.slots[li];
    if (LP == 32 && lane + 32 < A.e.L) sp1 = A.e.slots[lane + 32];
  }
  __syncthreads();
  if (blockIdx.x == 0) TRACE(31);
  uint32_t tab_s;
  asm volatile("mov.u32 %0, %1;" : "=r"(tab_s) : "r"(smem_u32(smem)));
  uint16_t* q = reinterpret_cast<uint16_t*>(smem + A.q_off) + wid * kTailQ;
  const int sh = 32 - V.log2n, bsh = 32 - V.log2B;
  const uint32_t nb = (uint32_t)V.nb, half = nb >> 1;
  const uint32_t half_s = half << sh;
  const int units = scnt[nenum];
  const int warp = blockIdx.x * (kTailNT / 32) + wid;
  const int nwarps = gridDim.x * (kTailNT / 32);
  for (int unit = warp; unit < units; unit += nwarps) {  // warp-uniform
    int e = 0;
    while (unit >= scnt[e + 1]) ++e;
    const int eq = V.pairs ? 2 * e : e;  // enumerated loop
    const uint32_t J = (uint32_t)__ldcg(V.Jp[eq] + (unit - scnt[e]));
    const uint32_t a = saa[eq];
    const uint32_t p0 = J * nb - half;  // first preimage of J (mod n via the scaled arithmetic below)
    // mandatory probes: pairs -> loop eq + 1; else loops e + 1 .. e + m with <= allowed misses
    const int m = V.pairs ? 1 : min(Lloc - V.T - e + 1, Lloc - 1 - e);
    const int allowed = V.pairs ? 0 : Lloc - V.T - e;
    for (uint32_t c0 = 0; c0 < nb; c0 += 32 * 32) {  // chunks of 32 candidates per lane
      const uint32_t P0 = (p0 + c0 + (uint32_t)lane) << sh;  // scaled position of the lane's first candidate
      const uint32_t lim = nb - c0;                          // candidates left in the unit
      uint32_t mask = 0u;
      if (V.pairs || m == 1) {
        const uint32_t qm = (uint32_t)eq + 1u;
        const uint32_t c = ssig[qm] * a;                     // sigma_q a_e: bucket of loop q from p
        const uint32_t bit = 1u << qm;
        uint32_t h = c * P0 + half_s;
        const uint32_t hs = c * (32u << sh);
        if (lim >= 32 * 32) {
#pragma unroll
          for (int i = 0; i < 32; ++i, h += hs)
            if (tab_at<ET>(tab_s, h >> bsh) & bit) mask |= 1u << i;
        } else {
          for (int i = 0; i < 32; ++i, h += hs)
            if ((uint32_t)(lane + 32 * i) < lim && (tab_at<ET>(tab_s, h >> bsh) & bit)) mask |= 1u << i;
        }
        if (!V.pairs && allowed >= 1) {  // m == 1 with a miss allowed: every candidate survives
          mask = 0u;
          for (int i = 0; i < 32; ++i)
            if ((uint32_t)(lane + 32 * i) < lim) mask |= 1u << i;
        }
      } else {
        for (int i = 0; i < 32; ++i) {
          if ((uint32_t)(lane + 32 * i) >= lim) break;
          const uint32_t Pi = P0 + ((32u * (uint32_t)i) << sh);
          const uint32_t F = a * Pi;
          int g = 0;
          for (int qq = 1; qq <= m; ++qq) {
            const int qd = e + qq;
            g += (tab_at<ET>(tab_s, (ssig[qd] * F + half_s) >> bsh) >> qd) & 1u;
          }
          if (m - g <= allowed) mask |= 1u << i;
        }
      }
      // compact the survivors into the warp's queue (u16 offsets inside the chunk)
      const int cnt = __popc(mask);
      const int incl = warp_incl_scan(cnt);
      const int total = __shfl_sync(kFull, incl, 31);
      int pos = incl - cnt;
      for (uint32_t mm = mask; mm; mm &= mm - 1) q[pos++] = (uint16_t)(lane + 32 * (__ffs(mm) - 1));
      __syncwarp();
      for (int b0 = 0; b0 < total; b0 += 32) {  // finish 32 survivors at a time
        bool hit = false;
        uint32_t f = 0u;
        if (b0 + lane < total) {
          const uint32_t F = a * ((p0 + c0 + (uint32_t)q[b0 + lane]) << sh);
          f = F >> sh;
          uint32_t bits = 0u;
          for (int qq = 0; qq < Lloc; ++qq) bits |= tab_at<ET>(tab_s, (ssig[qq] * F + half_s) >> bsh) & (1u << qq);
          if (V.pairs) {
            const uint32_t below = bits & ((1u << (2 * e)) - 1u);
            hit = __popc(bits) >= V.T && (below & (below >> 1) & 0x55555555u) == 0u;
          } else {
            hit = __popc(bits) >= V.T && (bits & ((1u << e) - 1u)) == 0u;
          }
        }
        tail_emit_estimate<LP>(A, hit, f, sp0, sp1);
      }
      __syncwarp();
    }
  }
  // ---- the last CTA to finish selects the output
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    s_last = atomicAdd(A.done, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (blockIdx.x == 0) TRACE(32);
  if (!s_last) return;
  __threadfence();
  output_body(smem, V.hits, V.hit_count, V.max_hits, A.e.hit_vals, A.e.hit_keys, A.e.out_hist, A.k, A.kp2, A.log2n,
              A.locs, A.vals, A.status);
}

}  // namespace cusfft
