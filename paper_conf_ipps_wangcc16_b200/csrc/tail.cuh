// tail.cuh — Steps 5 + 6 + output in ONE kernel (k_tail), after the cutoff:
//
//   Step 5  reverse hash + vote      PAPER.md:L91-L93, Alg. 4
//   Step 6  median estimation        PAPER.md:L95, Alg. 5
//   output  k strongest, by f        PAPER.md:L13 (k large coefficients), Alg. 5
//
// CTAs of 256 threads, several per SM.  Every CTA holds the location loops' cutoff
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
// Output: k_output (one CTA of 1024 threads, launched programmatically after
// k_tail) selects the k hits of largest |val|^2 (ties to the smaller f) and
// writes them sorted by f.
#pragma once
#include "exec_kernels.cuh"

namespace cusfft {

struct TailArgs {
  VoteArgs v;          // location loops in vote order: bitmaps, winner lists, sigma, a (pk: ET table or null)
  EstArgs e;           // every slot: records, slot params, 1/G^, phase tables, hit buffers, output-key histogram
  int q_off;           // byte offset of the per-warp queues in dynamic smem
};

constexpr int kTailNT = 256;  // threads per CTA (several CTAs per SM: a CTA waits only for its own 8 warps)
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
  const int tid = threadIdx.x, lane = tid & 31;
  CTRACE(80);
  // The first loads of the fast path are issued before the first barrier: the
  // hit count, the level-0 histogram (counted by the estimation; copied to
  // shared memory) and up to PF keys per thread, read speculatively below
  // max_hits and masked once H is known.  f and the value are loaded only for
  // the selected items.
  constexpr int PF = 4;  // fast path: H <= PF * 1024 items, kp2 <= 1024
  uint32_t* h0 = reinterpret_cast<uint32_t*>(smem + output_smem_bytes(kp2));
  double2* selv = reinterpret_cast<double2*>(ckey);  // [kp2] values of the selected entries (fast path)
  const unsigned hc = __ldcg(hit_count);
  uint32_t hb[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) hb[j] = __ldcg(ghist + tid + j * 1024);
  uint64_t pk[PF];
  uint32_t pf[PF];
  double2 pv[PF];
#pragma unroll
  for (int u = 0; u < PF; ++u) {
    const int i = u * 1024 + tid;
    if (i < max_hits) pk[u] = __ldcg(hit_keys + i);
  }
#pragma unroll
  for (int j = 0; j < 4; ++j) h0[tid + j * 1024] = hb[j];
  ghist = h0;
  const int H = min((int)hc, max_hits);
  if (tid == 0 && (int)hc > max_hits) atomicOr(status, 1);
  const int K = min(k, H);
  const bool fast = H <= PF * 1024 && kp2 <= 1024;
  if (tid == 0) sm[41] = 0;
  bcnt[tid] = 0;
  __syncthreads();
  CTRACE(81);
  bool direct = false;  // selv holds the values
  if (fast) {
    uint32_t d0 = 0;
    bool whole = true;
    if (H > K) {
      const BinPick b0 = pick_bin(ghist, K, sm);  // syncs
      d0 = (uint32_t)b0.d;
      whole = (K - b0.above) == b0.cnt;
    }
    CTRACE(82);
    if (whole) {  // the boundary bin is taken whole: selected = digit >= d0; positions by one block scan
      direct = true;
      bool take[PF];
      int cnt = 0;
#pragma unroll
      for (int u = 0; u < PF; ++u) {
        const int i = u * 1024 + tid;
        take[u] = i < H && ((uint32_t)(pk[u] >> 51) & 0xFFFu) >= d0;
        cnt += take[u];
        if (take[u]) {  // in flight across the scan's barriers
          pf[u] = (uint32_t)__ldcg(hits + i);
          pv[u] = __ldcg(hit_vals + i);
        }
      }
      int total;
      int pos = block_excl_scan<1024>(cnt, &total, sm);
#pragma unroll
      for (int u = 0; u < PF; ++u) {
        if (take[u]) {
          if (pos < kp2) {
            sel[pos] = ((uint64_t)pf[u] << 32) | (uint32_t)pos;
            selv[pos] = pv[u];
          }
          ++pos;
        }
      }
      if (tid == 0) sm[41] = total;
      __syncthreads();
    }
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
  CTRACE(83);
  const int ns = min(sm[41], kp2);
  if (tid == 0 && sm[41] != K) atomicOr(status + 2, 1);
  // bucket sort by the top 10 bits of f: an item's rank inside its bucket is
  // the counter value its atomic returns; one scan places the buckets
  const int sh = max(0, log2n - 10);
  int rnk[8];  // kp2 <= 8192: at most 8 items per thread
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    const int i = tid + u * 1024;
    if (i < ns) rnk[u] = atomicAdd(&bcnt[(int)(sel[i] >> 32) >> sh], 1);
  }
  __syncthreads();
  const int c = bcnt[tid];
  int total;
  const int st = block_excl_scan<1024>(c, &total, sm);
  bstart[tid] = st;
  const int cmax = __reduce_max_sync(kFull, c);
  if (tid == 0) sm[42] = 0;
  __syncthreads();
  if (lane == 0) atomicMax(&sm[42], cmax);
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    const int i = tid + u * 1024;
    if (i < ns) srt[bstart[(int)(sel[i] >> 32) >> sh] + rnk[u]] = sel[i];
  }
  __syncthreads();
  CTRACE(84);
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
  CTRACE(85);
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
  CTRACE(86);
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


// Step 6 for the hit each lane segment holds (frequency hf; valid = it
// exists).  LP = 16: a 16-lane segment per hit, lane li = slot li (L <= 16);
// LP = 32: one hit per warp, lanes hold slots li and li + 32 (L <= 64).
// Per-loop values stay in v0 / v1, the median in (vr, vi).  Warp-uniform.
template <int LP>
__device__ __forceinline__ void tail_estimate(const EstArgs& E, uint32_t hf, bool valid, const SlotParam& sp0,
                                              const SlotParam& sp1, double& vr, double& vi, double2& v0,
                                              double2& v1) {
  const int lane = threadIdx.x & 31;
  const int L = E.L;
  const int med = (L - 1) >> 1;
  const int seg = lane / LP, li = lane % LP;
  v0 = make_double2(0.0, 0.0);
  v1 = make_double2(0.0, 0.0);
  if (LP == 16) {
    const unsigned segmask = 0xFFFFu << (seg * 16);
    const bool act = li < L;
#ifdef CUSFFT_TRACE
    const long long te0 = clock64();
#endif
    if (valid && act) v0 = loop_estimate(E, sp0, li, hf);
#ifdef CUSFFT_TRACE
    {
      const bool nanv = v0.x != v0.x;  // waits for the loads
      const long long te1 = clock64();
      if (lane == 0 && valid) atomicMax(&g_trace[75], (unsigned long long)(te1 - te0 + (nanv ? 1 : 0)));
    }
#endif
#pragma unroll
    for (int part = 0; part < 2; ++part) {
      const double a = part ? v0.y : v0.x;
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
    if (valid) {
      if (lane < L) v0 = loop_estimate(E, sp0, lane, hf);
      if (lane + 32 < L) v1 = loop_estimate(E, sp1, lane + 32, hf);
    }
    vr = warp_rank_select(v0.x, v1.x, L, med);
    vi = warp_rank_select(v0.y, v1.y, L, med);
  }
}

// Results of tail_estimate for hit-list position hs (valid: hs < max_hits).
template <int LP>
__device__ __forceinline__ void tail_store(const EstArgs& E, unsigned hs, bool valid, double vr, double vi,
                                           const double2& v0, const double2& v1) {
  if (!valid) return;
  const int lane = threadIdx.x & 31;
  const int L = E.L, li = lane % LP;
  if (E.per_loop) {
    if (LP == 16) {
      if (li < L) E.per_loop[(int64_t)hs * L + li] = v0;
    } else {
      if (lane < L) E.per_loop[(int64_t)hs * L + lane] = v0;
      if (lane + 32 < L) E.per_loop[(int64_t)hs * L + lane + 32] = v1;
    }
  }
  if (li == 0) {
    const uint64_t key = (uint64_t)__double_as_longlong(__dadd_rn(__dmul_rn(vr, vr), __dmul_rn(vi, vi)));
    E.hit_vals[hs] = make_double2(vr, vi);
    E.hit_keys[hs] = key;
    atomicAdd(E.out_hist + ((uint32_t)(key >> 51) & 0xFFFu), 1u);
  }
}

// Hits of one finish round (hit: this lane's candidate is a hit, f its
// frequency): queued in the CTA's shared list (estimated by the whole CTA
// after its vote), or -- when that list is full -- given their hit-list
// positions and estimated by this warp at once.
constexpr int kTailHQ = 1024;  // CTA hit-queue capacity

template <int LP, bool EST>
__device__ __forceinline__ void tail_emit(const TailArgs& A, bool hit, uint32_t f, uint32_t* hq, int* nq,
                                          const SlotParam& sp0, const SlotParam& sp1) {
  const int lane = threadIdx.x & 31;
  const unsigned hb = __ballot_sync(kFull, hit);
  if (!hb) return;
  const int leader = __ffs(hb) - 1;
  const unsigned rank = __popc(hb & ((1u << lane) - 1u));
  int qpos = 0;
  if (lane == leader) qpos = atomicAdd(nq, __popc(hb));
  qpos = __shfl_sync(kFull, qpos, leader);
  if (qpos + __popc(hb) <= kTailHQ) {  // warp-uniform
    if (hit) hq[qpos + rank] = f;
    return;
  }
  if (lane == leader) atomicSub(nq, __popc(hb));  // overflow: this warp places and estimates them itself
  unsigned base = 0;
  if (lane == leader) base = atomicAdd(A.v.hit_count, (unsigned)__popc(hb));
  base = __shfl_sync(kFull, base, leader);
  const unsigned myslot = base + rank;
  if (hit && (int)myslot < A.v.max_hits) A.v.hits[myslot] = (int)f;
  if (!EST) return;
  constexpr int G = 32 / LP;
  unsigned rem = hb;
  while (rem) {  // warp-uniform
    int src[G];
#pragma unroll
    for (int g = 0; g < G; ++g) {
      src[g] = rem ? __ffs(rem) - 1 : -1;
      if (rem) rem &= rem - 1;
    }
    const int seg = lane / LP;
    int s = src[0];
#pragma unroll
    for (int g = 1; g < G; ++g)
      if (seg == g) s = src[g];
    const uint32_t hf = __shfl_sync(kFull, f, s < 0 ? 0 : s);
    const unsigned hs = __shfl_sync(kFull, myslot, s < 0 ? 0 : s);
    const bool valid = s >= 0 && (int)hs < A.v.max_hits;
    double vr, vi;
    double2 v0, v1;
    tail_estimate<LP>(A.e, hf, valid, sp0, sp1, vr, vi, v0, v1);
    tail_store<LP>(A.e, hs, valid, vr, vi, v0, v1);
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

// The vote table in global memory, built once from the location loops'
// cutoff bitmaps (plans whose cutoff cannot OR its winners into it directly:
// multi-GPU plans after the exchange); every k_tail CTA then bulk-copies it
// instead of transposing the bitmaps itself.  Thread per bucket.
template <typename ET>
__global__ void __launch_bounds__(256) k_pk_build(VoteArgs V, ET* __restrict__ pk) {
  pdl_wait();
  const int b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= V.B) return;
  uint32_t v = 0u;
  for (int q = 0; q < V.Lloc; ++q) v |= ((__ldcg(V.bmp[q] + (b >> 5)) >> (b & 31)) & 1u) << q;
  pk[b] = (ET)v;
}

// ET: vote table element; LP: estimation lanes per hit (16 or 32).
// LL: L_loc at compile time (8, the default plans) or 0 (any L_loc <= 8 sizeof(ET)).
// EST = false: the vote only (shard_mode 2, exchange.cuh: each rank estimates
// its own loops afterwards); the hits are written to the hit list unordered.
template <typename ET, int LP, int LL, bool EST = true>
__global__ void __launch_bounds__(kTailNT, 4) k_tail(TailArgs A) {
  pdl_wait();
  KTRACE(9);
  extern __shared__ __align__(16) uint8_t smem[];
  __shared__ uint32_t ssig[kMaxLoc], saa[kMaxLoc];
  __shared__ int scnt[kMaxLoc + 1];
  __shared__ int s_nq;
  __shared__ unsigned s_base;
  __shared__ uint32_t s_hq[kTailHQ];  // this CTA's hits (frequencies), estimated after its vote
  const VoteArgs& V = A.v;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  if (blockIdx.x == 0) TRACE(30);
  const int B = V.B, Lloc = V.Lloc;
  const int nenum = V.pairs ? Lloc / 2 : Lloc - V.T + 1;
  const int warp = blockIdx.x * (kTailNT / 32) + wid;
  // the warp's first winner bucket J, loaded now so its latency overlaps the table copy
  uint32_t Jpre = 0u;
  if (V.cnt_fixed && warp < nenum * V.num) {
    const int e0 = warp / V.num;
    Jpre = (uint32_t)__ldcg(V.Jp[V.pairs ? 2 * e0 : e0] + (warp - e0 * V.num));
  }
  // ---- the vote table: bulk-copied (the cutoff ORed the winners into V.pk) or transposed from the bitmaps
  __shared__ __align__(8) uint64_t tbar;
  const uint32_t tbytes = (uint32_t)(((int64_t)B * sizeof(ET) + 15) & ~int64_t(15));
  if (V.pk) {
    if (tid == 0) {
      mbar_init(&tbar, 1);
      mbar_expect_tx(&tbar, tbytes);
      for (uint32_t o = 0; o < tbytes; o += 32768u)
        bulk_g2s(smem + o, reinterpret_cast<const uint8_t*>(V.pk) + o, min(32768u, tbytes - o), &tbar,
                 l2_policy_last());
    }
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
  if (tid < Lloc) {
    ssig[tid] = V.sig[tid];
    saa[tid] = V.aa[tid];
  }
  // unit prefix over the enumerated loops' winner counts (exactly num each
  // unless Alg. 6's threshold cutoff ran: then loaded in parallel, summed by one thread)
  if (tid < nenum) scnt[tid + 1] = V.cnt_fixed ? V.num : __ldcg(V.cntp[V.pairs ? 2 * tid : tid]);
  if (tid == 0) s_nq = 0;
  __syncthreads();
  if (tid == 0) {
    scnt[0] = 0;
    for (int e = 0; e < nenum; ++e) scnt[e + 1] += scnt[e];
  }
  // slot parameters of the lanes' estimation slots
  SlotParam sp0{0, 0, 0, 0}, sp1{0, 0, 0, 0};
  {
    const int li = LP == 16 ? (lane & 15) : lane;
    if (li < A.e.L) sp0 = A.e.slots[li];
    if (LP == 32 && lane + 32 < A.e.L) sp1 = A.e.slots[lane + 32];
  }
  __syncthreads();
  if (V.pk) mbar_wait(&tbar, 0);
  if (blockIdx.x == 0) TRACE(31);
#ifdef CUSFFT_TRACE
  const long long c_vote0 = clock64();
#endif
  uint32_t tab_s;
  asm volatile("mov.u32 %0, %1;" : "=r"(tab_s) : "r"(smem_u32(smem)));
  uint16_t* q = reinterpret_cast<uint16_t*>(smem + A.q_off) + wid * kTailQ;
  const int sh = 32 - V.log2n, bsh = 32 - V.log2B;
  const uint32_t nb = (uint32_t)V.nb, half = nb >> 1;
  const uint32_t half_s = half << sh;
  const int units = scnt[nenum];
  const int nwarps = gridDim.x * (kTailNT / 32);
  for (int unit = warp; unit < units; unit += nwarps) {  // warp-uniform
    int e = 0;
    while (unit >= scnt[e + 1]) ++e;
    const int eq = V.pairs ? 2 * e : e;  // enumerated loop
    const uint32_t J = (V.cnt_fixed && unit == warp) ? Jpre : (uint32_t)__ldcg(V.Jp[eq] + (unit - scnt[e]));
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
          if (LL > 0) {  // compile-time L_loc: unrolled (sigmas by broadcast shared loads)
#pragma unroll
            for (int qq = 0; qq < (LL > 0 ? LL : 1); ++qq)
              bits |= tab_at<ET>(tab_s, (ssig[qq] * F + half_s) >> bsh) & (1u << qq);
          } else {
            for (int qq = 0; qq < Lloc; ++qq) bits |= tab_at<ET>(tab_s, (ssig[qq] * F + half_s) >> bsh) & (1u << qq);
          }
          if (V.pairs) {
            const uint32_t below = bits & ((1u << (2 * e)) - 1u);
            hit = __popc(bits) >= V.T && (below & (below >> 1) & 0x55555555u) == 0u;
          } else {
            hit = __popc(bits) >= V.T && (bits & ((1u << e) - 1u)) == 0u;
          }
        }
        tail_emit<LP, EST>(A, hit, f, s_hq, &s_nq, sp0, sp1);
      }
      __syncwarp();
    }
  }
  // ---- Step 6 for this CTA's queued hits: one block of hit-list positions,
  // then 32 / LP hits per warp per pass
  pdl_launch_dependents();  // the output kernel may become resident as CTAs drain
  TRACE_END(33);  // (trace builds) latest end of a CTA's vote
#ifdef CUSFFT_TRACE
  CTRACE_MAX(70, clock64() - c_vote0);  // longest warp-0 vote (cycles)
#endif
  // (the first pass is computed while thread 0's reservation of hit-list
  // positions is in flight; it is stored once the base is known)
  __syncthreads();
#ifdef CUSFFT_TRACE
  const long long c_est0 = clock64();
  CTRACE_MAX(71, c_est0 - c_vote0);  // longest CTA vote incl. its barrier (cycles)
#endif
  const int nq = s_nq;
  if (tid == 0 && nq > 0) s_base = atomicAdd(V.hit_count, (unsigned)nq);
  if (!EST) {
    __syncthreads();
    const unsigned base = s_base;
    for (int i = tid; i < nq; i += kTailNT)
      if ((int)(base + i) < V.max_hits) V.hits[base + i] = (int)s_hq[i];
    return;
  }
  constexpr int G = 32 / LP;
  constexpr int PASS = (kTailNT / 32) * G;  // hits per CTA pass
  const int h1 = wid * G + lane / LP;
  double vr = 0.0, vi = 0.0;
  double2 v0, v1;
  if (wid * G < nq)  // warp-uniform
    tail_estimate<LP>(A.e, h1 < nq ? s_hq[h1] : 0u, h1 < nq, sp0, sp1, vr, vi, v0, v1);
#ifdef CUSFFT_TRACE
  if (wid * G < nq && lane == 0) atomicMax(&g_trace[73], (unsigned long long)(clock64() - c_est0));  // first pass estimated
#endif
  __syncthreads();
#ifdef CUSFFT_TRACE
  CTRACE_MAX(74, clock64() - c_est0);  // + the block barrier (hit-list base known)
#endif
  if (nq > 0) {
    const unsigned base = s_base;
    for (int i = tid; i < nq; i += kTailNT)
      if ((int)(base + i) < V.max_hits) V.hits[base + i] = (int)s_hq[i];
    if (wid * G < nq) tail_store<LP>(A.e, base + (unsigned)h1, h1 < nq && (int)(base + h1) < V.max_hits, vr, vi, v0, v1);
    for (int hh = wid * G + PASS; hh < nq; hh += PASS) {  // more than one pass of hits (warp-uniform)
      const int h = hh + lane / LP;
      tail_estimate<LP>(A.e, h < nq ? s_hq[h] : 0u, h < nq, sp0, sp1, vr, vi, v0, v1);
      tail_store<LP>(A.e, base + (unsigned)h, h < nq && (int)(base + h) < V.max_hits, vr, vi, v0, v1);
    }
  }
  TRACE_END(34);  // (trace builds) latest end of a CTA's estimation
#ifdef CUSFFT_TRACE
  CTRACE_MAX(72, clock64() - c_est0);  // longest CTA estimation (cycles)
#endif
}

}  // namespace cusfft
