// exec_kernels.cuh — the timed hot path:
//   k_fold      Steps 1+2  permutation + filter + fold into B buckets
//   k_fft       Step 3     batched B-point FFT (fft.cuh; one or two passes)
//   k_select    Step 4     exact top-num cutoff per location loop
//   k_vote      Step 5     reverse hash + vote
//   k_estimate  Step 6     per-loop estimates and their median
//   k_output    output     top-k hits by |val|^2, sorted by location
#pragma once
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
__device__ __forceinline__ double2 ld_gather(const double2* p) {
  double2 v;
  asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  return v;
}

template <int RC>
__global__ void __launch_bounds__(256) k_fold(const double2* __restrict__ x, const double* __restrict__ taps,
                                              const SlotParam* __restrict__ slots, double2* __restrict__ u,
                                              int B, int w, int R, uint32_t nmask) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x;
  const int s = blockIdx.y;
  if (j >= B) return;
  const uint32_t sigma = slots[s].sigma, tau = slots[s].tau;
  double ar = 0.0, ai = 0.0;
  for (int r0 = 0; r0 < R; r0 += RC) {
    double2 v[RC];
    double g[RC];
#pragma unroll
    for (int c = 0; c < RC; ++c) {
      const int i = j + (r0 + c) * B;
      if (r0 + c < R && i < w) {
        const uint32_t idx = (sigma * (uint32_t)i + tau) & nmask;  // mod n, n | 2^32
        v[c] = ld_gather(x + idx);
        g[c] = __ldg(taps + i);
      }
    }
#pragma unroll
    for (int c = 0; c < RC; ++c) {
      const int i = j + (r0 + c) * B;
      if (r0 + c < R && i < w) {
        ar = __dadd_rn(ar, __dmul_rn(g[c], v[c].x));
        ai = __dadd_rn(ai, __dmul_rn(g[c], v[c].y));
      }
    }
  }
  u[(size_t)s * B + j] = make_double2(ar, ai);
}

// ---------------------------------------------------------------------------
// Record layout of one slot in the exchange buffer:
//   [u^ : B x double2][bitmap : B/32 x u32][J : num x int32], 256-B aligned.
// ---------------------------------------------------------------------------
struct RecLayout {
  int64_t rec_bytes, off_bitmap, off_J;
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

// ---------------------------------------------------------------------------
// Step 4 (L89, Alg. 3; the linear-time selection of §V.B,
// made exact): J_r = the num buckets of largest |u^|^2 = re*re + im*im, ties
// to the smaller bucket, as a bitmap and an ascending list.  One CTA of 1024
// threads per location slot of this rank.
//  1. the FFT epilogue already counted keys per top-12-bit digit: a block scan
//     of that histogram gives the boundary digit d0 and the count above it;
//  2. one pass over the B keys: digit > d0 -> selected, digit == d0 -> smem
//     candidate list;
//  3. exact 96-bit radix select (key, ~bucket) among the candidates.
// Falls back to a full radix select over all keys when the boundary bin holds
// more than kSelCap candidates.  Resets the histogram for the next execution.
// Dynamic smem: 4096 u32 hist + 64 int + kSelCap x (u64 + int).
// ---------------------------------------------------------------------------
constexpr int kSelCap = 4096;

__global__ void __launch_bounds__(1024) k_select(uint8_t* __restrict__ records, RecLayout lay,
                                                 const int* __restrict__ sel_slots, int B, int num,
                                                 const uint64_t* __restrict__ gkeys, uint32_t* __restrict__ ghist,
                                                 int* __restrict__ status) {
  extern __shared__ __align__(16) uint8_t smem[];
  uint32_t* hist = reinterpret_cast<uint32_t*>(smem);
  int* sm = reinterpret_cast<int*>(smem + 4096 * 4);
  uint64_t* ckey = reinterpret_cast<uint64_t*>(smem + 4096 * 4 + 64 * 4);
  int* cidx = reinterpret_cast<int*>(ckey + kSelCap);
  const int tid = threadIdx.x;
  const int sel = blockIdx.x;
  uint8_t* rec = records + (int64_t)sel_slots[sel] * lay.rec_bytes;
  uint32_t* bitmap = reinterpret_cast<uint32_t*>(rec + lay.off_bitmap);
  int* J = reinterpret_cast<int*>(rec + lay.off_J);
  const uint64_t* keys = gkeys + (int64_t)sel * B;
  uint32_t* gh = ghist + (int64_t)sel * 4096;
  const int words = (B + 31) >> 5;

  // 1. boundary digit from the histogram (thread t owns bins 4095-4t .. 4092-4t)
  const int base = 4095 - 4 * tid;
  const int c0 = gh[base], c1 = gh[base - 1], c2 = gh[base - 2], c3 = gh[base - 3];
  const int mine = c0 + c1 + c2 + c3;
  int total;
  const int ex = block_excl_scan<1024>(mine, &total, sm);
  if (ex < num && num <= ex + mine) {
    int cum = ex, d, cnt;
    if (cum + c0 >= num) {
      d = base; cnt = c0;
    } else if ((cum += c0) + c1 >= num) {
      d = base - 1; cnt = c1;
    } else if ((cum += c1) + c2 >= num) {
      d = base - 2; cnt = c2;
    } else {
      cum += c2; d = base - 3; cnt = c3;
    }
    sm[32] = d; sm[33] = cum; sm[34] = cnt;
  }
  gh[base] = 0; gh[base - 1] = 0; gh[base - 2] = 0; gh[base - 3] = 0;  // self-reset
  for (int w = tid; w < words; w += 1024) bitmap[w] = 0;
  if (tid == 0) sm[40] = 0;
  __syncthreads();
  const uint32_t d0 = (uint32_t)sm[32];
  const int above = sm[33], cnt0 = sm[34];
  const int k2 = num - above;  // 1 <= k2 <= cnt0
  const bool whole_bin = (k2 == cnt0);
  // 2. one pass over the keys, 16 loads in flight per thread
  for (int i0 = 0; i0 < B; i0 += 16 * 1024) {
    uint64_t kb[16];
#pragma unroll
    for (int u = 0; u < 16; ++u) {
      const int i = i0 + u * 1024 + tid;
      kb[u] = i < B ? __ldg(keys + i) : 0ull;
    }
#pragma unroll
    for (int u = 0; u < 16; ++u) {
      const int i = i0 + u * 1024 + tid;
      if (i >= B) continue;
      const uint32_t d = (uint32_t)(kb[u] >> 51) & 0xFFFu;
      if (d > d0 || (d == d0 && whole_bin)) {
        atomicOr(&bitmap[i >> 5], 1u << (i & 31));
      } else if (d == d0) {
        const int pos = atomicAdd(&sm[40], 1);
        if (pos < kSelCap) {
          ckey[pos] = kb[u];
          cidx[pos] = i;
        }
      }
    }
  }
  __syncthreads();
  if (!whole_bin) {
    const int nc = sm[40];
    if (nc <= kSelCap) {
      const Prefix96 p = block_radix_select(PairSrc{ckey, cidx}, nc, k2, hist, sm);
      for (int c = tid; c < nc; c += 1024)
        if (ge96(p, ckey[c], ~(uint32_t)cidx[c])) atomicOr(&bitmap[cidx[c] >> 5], 1u << (cidx[c] & 31));
    } else {  // crowded boundary bin: exact select over all keys
      const Prefix96 p = block_radix_select(KeysSrc{keys}, B, num, hist, sm);
      for (int w = tid; w < words; w += 1024) {
        uint32_t bits = 0;
        for (int b = 0; b < 32; ++b) {
          const int i = w * 32 + b;
          if (i < B && ge96(p, keys[i], ~(uint32_t)i)) bits |= 1u << b;
        }
        bitmap[w] = bits;
      }
    }
  }
  __syncthreads();
  // 3. ascending winner list from the bitmap
  const int wpt = (words + 1023) >> 10;
  int cnt = 0;
  for (int w = tid * wpt; w < min(words, (tid + 1) * wpt); ++w) cnt += __popc(bitmap[w]);
  int pos = block_excl_scan<1024>(cnt, &total, sm);
  for (int w = tid * wpt; w < min(words, (tid + 1) * wpt); ++w) {
    uint32_t bits = bitmap[w];
    while (bits) {
      const int b = __ffs(bits) - 1;
      bits &= bits - 1;
      if (pos < num) J[pos] = w * 32 + b;
      ++pos;
    }
  }
  if (tid == 0 && total != num) atomicOr(status + 1, 1);
}

// ---------------------------------------------------------------------------
// Step 5 (L91-L93, Alg. 4).  bucket_q(f) = ((sigma_q f + nb/2) mod n) / nb
// is Alg. 4's range [ceil((J-1/2) nb), ceil((J+1/2) nb)).  A frequency with
// >= T of L_loc votes is selected in at least one of the first L_loc - T + 1
// location loops, so candidates f = a_{q0} p are enumerated only from those
// loops' preimage ranges, and f is counted at the first loop q0 that selects
// it: it needs T-1 votes among the loops after q0 (probed first: a random
// candidate is rejected after L_loc - T - q0 + 1 misses) and no vote before
// q0 (probed last, for the rare survivors).
// Dynamic smem: L_loc * ceil(B/32) u32 bitmaps.
// ---------------------------------------------------------------------------
struct VoteArgs {
  const uint8_t* records;
  RecLayout lay;
  const int* loc_slots;  // [L_loc] slot of each location loop, in vote order
  const uint32_t* loc_sigma;
  const uint32_t* loc_a;
  int Lloc, T, num, B, nb, log2nb, P, log2P;
  uint32_t nmask;
  int* hits;
  unsigned* hit_count;
  int max_hits;
};

__global__ void __launch_bounds__(256) k_vote(VoteArgs A) {
  extern __shared__ __align__(16) uint8_t smem[];
  uint32_t* bm = reinterpret_cast<uint32_t*>(smem);
  __shared__ uint32_t ssig[64];
  const int words = (A.B + 31) >> 5;
  if ((words & 3) == 0) {  // 16-B vector loads, 8 in flight per thread
    const int v4 = words >> 2, tot = A.Lloc * v4;
    uint4* bm4 = reinterpret_cast<uint4*>(bm);
    for (int i0 = 0; i0 < tot; i0 += 8 * (int)blockDim.x) {
      uint4 tmp[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int i = i0 + u * blockDim.x + threadIdx.x;
        if (i < tot) {
          const int q = i / v4, w = i - q * v4;
          tmp[u] = __ldg(reinterpret_cast<const uint4*>(A.records + (int64_t)A.loc_slots[q] * A.lay.rec_bytes +
                                                        A.lay.off_bitmap) + w);
        }
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int i = i0 + u * blockDim.x + threadIdx.x;
        if (i < tot) bm4[i] = tmp[u];
      }
    }
  } else {
    for (int q = 0; q < A.Lloc; ++q) {
      const uint32_t* src = reinterpret_cast<const uint32_t*>(A.records + (int64_t)A.loc_slots[q] * A.lay.rec_bytes +
                                                               A.lay.off_bitmap);
      for (int i = threadIdx.x; i < words; i += blockDim.x) bm[q * words + i] = src[i];
    }
  }
  if (threadIdx.x < A.Lloc) ssig[threadIdx.x] = A.loc_sigma[threadIdx.x];
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int log_cpj = A.log2nb - A.log2P;  // chunks per bucket = nb / P
  const int per_q = A.num << log_cpj;
  const int items = (A.Lloc - A.T + 1) * per_q;
  const uint32_t half = (uint32_t)(A.nb >> 1);
  const int stride = gridDim.x * blockDim.x;
  const int warp_start = blockIdx.x * blockDim.x + threadIdx.x - lane;
  for (int it0 = warp_start; it0 < items; it0 += stride) {
    const int it = it0 + lane;
    const bool valid_item = it < items;
    int q0 = 0;
    uint32_t a = 0, p = 0;
    if (valid_item) {
      q0 = it / per_q;
      const int rem = it - q0 * per_q;
      const int jidx = rem >> log_cpj;
      const int chunk = rem & ((1 << log_cpj) - 1);
      const int* Jl = reinterpret_cast<const int*>(A.records + (int64_t)A.loc_slots[q0] * A.lay.rec_bytes +
                                                   A.lay.off_J);
      const uint32_t Jv = (uint32_t)Jl[jidx];
      p = (Jv * (uint32_t)A.nb - half + (uint32_t)(chunk * A.P)) & A.nmask;
      a = A.loc_a[q0];
    }
    const int allowed = A.Lloc - A.T - q0;
    uint32_t f = (a * p) & A.nmask;
    for (int t = 0; t < A.P; ++t, f = (f + a) & A.nmask) {
      bool hit = false;
      if (valid_item) {
        int miss = 0;
        bool ok = true;
        for (int q = q0 + 1; q < A.Lloc; ++q) {
          const uint32_t b = ((ssig[q] * f + half) & A.nmask) >> A.log2nb;
          if (!((bm[q * words + (b >> 5)] >> (b & 31)) & 1u) && ++miss > allowed) {
            ok = false;
            break;
          }
        }
        if (ok) {
          for (int q = 0; q < q0; ++q) {
            const uint32_t b = ((ssig[q] * f + half) & A.nmask) >> A.log2nb;
            if ((bm[q * words + (b >> 5)] >> (b & 31)) & 1u) {
              ok = false;
              break;
            }
          }
        }
        hit = ok;
      }
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
  }
}

// ---------------------------------------------------------------------------
// Step 6 (L95, Alg. 5), one warp per hit, one lane per loop (slot).
// For hit f and loop l:  p = sigma_l f mod n, h = p / nb, d = p mod nb;
//   if d > nb/2: h = h+1 mod B, d -= nb;
//   v_l = u^_l[h] * e^{-2 pi i tau_l f / n} / G^(-d);
// val = (element of rank (L-1)/2 of Re v) + i (same of Im v), ties by loop.
// ---------------------------------------------------------------------------
struct EstArgs {
  const uint8_t* records;
  RecLayout lay;
  const SlotParam* slots;
  int L;
  const double2* ghat;
  const int* hits;
  const unsigned* hit_count;
  int max_hits;
  uint32_t nmask;
  int log2nb, nb, B;
  double n;
  double2* hit_vals;
  uint64_t* hit_keys;
  double2* per_loop;  // may be null
};

constexpr int kMaxLoops = 64;

__device__ __forceinline__ double2 loop_estimate(const EstArgs& A, int l, uint32_t f) {
  const SlotParam sp = A.slots[l];
  const uint32_t p = (sp.sigma * f) & A.nmask;
  int hb = (int)(p >> A.log2nb);
  int d = (int)(p & (uint32_t)(A.nb - 1));
  if (d > (A.nb >> 1)) {
    hb = (hb + 1) & (A.B - 1);
    d -= A.nb;
  }
  const double2 g = __ldg(A.ghat + (A.nb >> 1) - d);  // G^(-d)
  const double2 b = reinterpret_cast<const double2*>(A.records + (int64_t)l * A.lay.rec_bytes)[hb];
  const uint32_t tph = (sp.tau * f) & A.nmask;
  double sn, cs;
  sincospi(2.0 * (double)tph / A.n, &sn, &cs);
  const double zr = b.x * cs + b.y * sn;  // b * e^{-i phi}
  const double zi = b.y * cs - b.x * sn;
  const double den = g.x * g.x + g.y * g.y;
  return make_double2((zr * g.x + zi * g.y) / den, (zi * g.x - zr * g.y) / den);
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
  const int H = min((int)*A.hit_count, A.max_hits);
  const int lane = threadIdx.x & 31;
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nwarps = (gridDim.x * blockDim.x) >> 5;
  const int med = (A.L - 1) >> 1;
  for (int h = warp; h < H; h += nwarps) {
    const uint32_t f = (uint32_t)A.hits[h];
    double2 v0 = make_double2(0.0, 0.0), v1 = make_double2(0.0, 0.0);
    if (lane < A.L) v0 = loop_estimate(A, lane, f);
    if (lane + 32 < A.L) v1 = loop_estimate(A, lane + 32, f);
    if (A.per_loop) {
      if (lane < A.L) A.per_loop[(int64_t)h * A.L + lane] = v0;
      if (lane + 32 < A.L) A.per_loop[(int64_t)h * A.L + lane + 32] = v1;
    }
    const double vr = warp_rank_select(v0.x, v1.x, A.L, med);
    const double vi = warp_rank_select(v0.y, v1.y, A.L, med);
    if (lane == 0) {
      A.hit_vals[h] = make_double2(vr, vi);
      A.hit_keys[h] = (uint64_t)__double_as_longlong(__dadd_rn(__dmul_rn(vr, vr), __dmul_rn(vi, vi)));
    }
  }
}

// ---------------------------------------------------------------------------
// Output: the k hits of largest |val|^2 (ties to the smaller f), written in
// ascending f; pads loc = -1, val = 0.  One CTA of 1024 threads.  Hits are
// staged in smem when H <= kOutCap; the sort is a bitonic network (warp
// shuffles below stride 32) over 64-bit (f << 32 | hit index) keys.
// Dynamic smem: 4096 u32 hist + 64 ints + kOutCap x (u64 + int) + kp2 x u64.
// ---------------------------------------------------------------------------
constexpr int kOutCap = 8192;

struct HitSrc {
  const uint64_t* keys;
  const int* hits;
  __device__ __forceinline__ void get(int i, uint64_t& hi, uint32_t& lo) const {
    hi = keys[i];
    lo = ~(uint32_t)hits[i];
  }
};

__global__ void __launch_bounds__(1024) k_output(const int* __restrict__ hits, const unsigned* __restrict__ hit_count,
                                                 int max_hits, const double2* __restrict__ hit_vals,
                                                 const uint64_t* __restrict__ hit_keys, int k, int kp2,
                                                 int64_t* __restrict__ locs, double2* __restrict__ vals,
                                                 int* __restrict__ status) {
  extern __shared__ __align__(16) uint8_t smem[];
  uint32_t* hist = reinterpret_cast<uint32_t*>(smem);
  int* sm = reinterpret_cast<int*>(smem + 4096 * 4);
  uint64_t* skey = reinterpret_cast<uint64_t*>(smem + 4096 * 4 + 64 * 4);
  int* shit = reinterpret_cast<int*>(skey + kOutCap);
  uint64_t* sort = reinterpret_cast<uint64_t*>(shit + kOutCap);
  const int tid = threadIdx.x;
  const unsigned hc = *hit_count;
  const int H = min((int)hc, max_hits);
  if (tid == 0 && (int)hc > max_hits) atomicOr(status, 1);
  const int K = min(k, H);
  const bool staged = H <= kOutCap;
  if (staged) {
    for (int i = tid; i < H; i += 1024) {
      skey[i] = hit_keys[i];
      shit[i] = hits[i];
    }
  }
  if (tid == 0) sm[40] = 0;
  for (int i = tid; i < kp2; i += 1024) sort[i] = ~0ull;
  __syncthreads();
  const uint64_t* kk = staged ? skey : hit_keys;
  const int* hh = staged ? shit : hits;
  Prefix96 p{0, 0, 0, 0};  // matches everything
  if (H > K) p = block_radix_select(HitSrc{kk, hh}, H, K, hist, sm);
  for (int i = tid; i < H; i += 1024) {
    const int f = hh[i];
    if (ge96(p, kk[i], ~(uint32_t)f)) {
      const int pos = atomicAdd(&sm[40], 1);
      if (pos < kp2) sort[pos] = ((uint64_t)(uint32_t)f << 32) | (uint32_t)i;
    }
  }
  __syncthreads();
  if (tid == 0 && sm[40] != K) atomicOr(status + 2, 1);
  if (kp2 <= 1024) {
    uint64_t v = tid < kp2 ? sort[tid] : ~0ull;
    for (int size = 2; size <= kp2; size <<= 1) {
      for (int stride = size >> 1; stride > 0; stride >>= 1) {
        uint64_t o;
        if (stride >= 32) {
          __syncthreads();
          sort[tid] = v;
          __syncthreads();
          o = sort[tid ^ stride];
        } else {
          o = __shfl_xor_sync(kFull, v, stride);
        }
        const bool up = (tid & size) == 0;
        const bool lower = (tid & stride) == 0;
        v = (lower == up) ? min(v, o) : max(v, o);
      }
    }
    __syncthreads();
    if (tid < kp2) sort[tid] = v;
    __syncthreads();
  } else {
    for (int size = 2; size <= kp2; size <<= 1) {
      for (int stride = size >> 1; stride > 0; stride >>= 1) {
        for (int t = tid; t < (kp2 >> 1); t += 1024) {
          const int i = 2 * t - (t & (stride - 1));
          const int jn = i + stride;
          const bool up = (i & size) == 0;
          const uint64_t a = sort[i], b = sort[jn];
          if ((a > b) == up) {
            sort[i] = b;
            sort[jn] = a;
          }
        }
        __syncthreads();
      }
    }
  }
  for (int j = tid; j < k; j += 1024) {
    if (j < K) {
      const uint64_t v = sort[j];
      locs[j] = (int64_t)(v >> 32);
      vals[j] = hit_vals[(uint32_t)v];
    } else {
      locs[j] = -1;
      vals[j] = make_double2(0.0, 0.0);
    }
  }
}

}  // namespace cusfft
