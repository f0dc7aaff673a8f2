// exec_kernels.cuh — the timed hot path:
//   k_fold      Steps 1+2  permutation + filter + fold into B buckets
//   k_fft_pass  Step 3     batched B-point FFT (one or two smem passes)
//   k_select    Step 4     exact top-num cutoff per location loop
//   k_vote      Step 5     reverse hash + vote
//   k_estimate  Step 6     per-loop estimates and their median
//   k_output    output     top-k hits by |val|^2, sorted by location
#pragma once
#include "common.cuh"

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
// Step 3 (L87, batched over loops as in L232): one pass of a four-step FFT.
// A CTA transforms NSEQ sequences of length m = 2^logm held in shared memory
// (radix-2 DIT after a bit-reversed load).  Sequence q = (slot l, column col):
//   element e at in [l*in_ls + col*in_cs + e*in_es],
//   result  e at out[l*out_ls + col*out_cs + e*out_es],
// optionally multiplied by tw[(col * e) mod B] = e^{-2 pi i col e / B}.
// Pass 1 (B = B1 B2, m = B1): in_cs = 1, in_es = B2, twiddle on.
// Pass 2 (m = B2): in_cs = B2, in_es = 1, out_cs = 1, out_es = B1.
// A single pass (B1 = 1) is a plain B-point FFT per slot.
// ---------------------------------------------------------------------------
constexpr int kFftSmemElems = 2048;

__global__ void __launch_bounds__(256) k_fft_pass(const double2* __restrict__ in, double2* __restrict__ out,
                                                  const double2* __restrict__ tw, int B, int logm, int nseq_cta,
                                                  int seq_per_slot, int total_seq, int64_t in_ls, int in_cs,
                                                  int in_es, int64_t out_ls, int out_cs, int out_es, int twiddle) {
  __shared__ double2 S[kFftSmemElems];
  const int m = 1 << logm;
  const int q0 = blockIdx.x * nseq_cta;
  const int nelem = nseq_cta * m;
  // load (coalesced along whichever stride is 1), bit-reversed into smem
  const bool col_fast_in = (in_cs == 1);
  for (int t = threadIdx.x; t < nelem; t += blockDim.x) {
    int sq, e;
    if (col_fast_in) {
      sq = t % nseq_cta;
      e = t / nseq_cta;
    } else {
      sq = t / m;
      e = t % m;
    }
    const int q = q0 + sq;
    if (q < total_seq) {
      const int l = q / seq_per_slot, col = q % seq_per_slot;
      const int rev = logm ? (int)(__brev((unsigned)e) >> (32 - logm)) : 0;
      S[sq * m + rev] = in[(int64_t)l * in_ls + (int64_t)col * in_cs + (int64_t)e * in_es];
    }
  }
  __syncthreads();
  const int twstride0 = B >> 1;  // tw index step for len = 2
  for (int s = 1; s <= logm; ++s) {
    const int half = 1 << (s - 1);
    const int tstride = twstride0 >> (s - 1);  // B / len
    for (int bf = threadIdx.x; bf < (nelem >> 1); bf += blockDim.x) {
      const int sq = bf >> (logm - 1);
      const int k = bf & ((m >> 1) - 1);
      const int pos = k & (half - 1);
      const int i0 = ((k >> (s - 1)) << s) + pos;
      const int i1 = i0 + half;
      const double2 wv = tw[pos * tstride];
      const double2 a = S[sq * m + i0];
      const double2 b = S[sq * m + i1];
      const double2 bw = make_double2(b.x * wv.x - b.y * wv.y, b.x * wv.y + b.y * wv.x);
      S[sq * m + i0] = make_double2(a.x + bw.x, a.y + bw.y);
      S[sq * m + i1] = make_double2(a.x - bw.x, a.y - bw.y);
    }
    __syncthreads();
  }
  const bool col_fast_out = (out_cs == 1);
  for (int t = threadIdx.x; t < nelem; t += blockDim.x) {
    int sq, e;
    if (col_fast_out) {
      sq = t % nseq_cta;
      e = t / nseq_cta;
    } else {
      sq = t / m;
      e = t % m;
    }
    const int q = q0 + sq;
    if (q < total_seq) {
      const int l = q / seq_per_slot, col = q % seq_per_slot;
      double2 v = S[sq * m + e];
      if (twiddle) {
        const double2 wv = tw[((int64_t)col * e) & (B - 1)];
        v = make_double2(v.x * wv.x - v.y * wv.y, v.x * wv.y + v.y * wv.x);
      }
      out[(int64_t)l * out_ls + (int64_t)col * out_cs + (int64_t)e * out_es] = v;
    }
  }
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

// Step 4 (L89, Alg. 3): J_r = the num buckets of largest
// |u^|^2 = re*re + im*im (ties to the smaller bucket), as a bitmap and as an
// ascending list.  One CTA of 1024 threads per location slot of this rank.
// Dynamic smem: 4096 u32 histogram + 64 ints + (keys_in_smem ? B u64 : 0).
__global__ void __launch_bounds__(1024) k_select(uint8_t* __restrict__ records, RecLayout lay,
                                                 const int* __restrict__ sel_slots, int B, int num,
                                                 uint64_t* __restrict__ gkeys, int keys_in_smem,
                                                 int* __restrict__ status) {
  extern __shared__ __align__(16) uint8_t smem[];
  uint32_t* hist = reinterpret_cast<uint32_t*>(smem);
  int* sm = reinterpret_cast<int*>(smem + 4096 * 4);
  uint64_t* skeys = reinterpret_cast<uint64_t*>(smem + 4096 * 4 + 64 * 4);
  const int slot = sel_slots[blockIdx.x];
  uint8_t* rec = records + (int64_t)slot * lay.rec_bytes;
  const double2* uhat = reinterpret_cast<const double2*>(rec);
  uint32_t* bitmap = reinterpret_cast<uint32_t*>(rec + lay.off_bitmap);
  int* J = reinterpret_cast<int*>(rec + lay.off_J);
  uint64_t* keys = keys_in_smem ? skeys : gkeys + (int64_t)blockIdx.x * B;
  for (int i = threadIdx.x; i < B; i += blockDim.x) {
    const double2 v = uhat[i];
    const double m2 = __dadd_rn(__dmul_rn(v.x, v.x), __dmul_rn(v.y, v.y));
    keys[i] = (uint64_t)__double_as_longlong(m2);
  }
  __syncthreads();
  const Prefix96 p = block_radix_select(KeysSrc{keys}, B, num, hist, sm);
  // bitmap words: thread t owns words [t*wpt, (t+1)*wpt)
  const int words = (B + 31) >> 5;
  const int wpt = (words + 1023) >> 10;
  int cnt = 0;
  for (int wi = threadIdx.x * wpt; wi < min(words, (threadIdx.x + 1) * wpt); ++wi) {
    uint32_t bits = 0;
    for (int b = 0; b < 32; ++b) {
      const int i = wi * 32 + b;
      if (i < B && ge96(p, keys[i], ~(uint32_t)i)) bits |= 1u << b;
    }
    bitmap[wi] = bits;
    cnt += __popc(bits);
  }
  int total;
  int pos = block_excl_scan<1024>(cnt, &total, sm);
  for (int wi = threadIdx.x * wpt; wi < min(words, (threadIdx.x + 1) * wpt); ++wi) {
    uint32_t bits = bitmap[wi];
    while (bits) {
      const int b = __ffs(bits) - 1;
      bits &= bits - 1;
      if (pos < num) J[pos] = wi * 32 + b;
      ++pos;
    }
  }
  if (threadIdx.x == 0 && total != num) atomicOr(status + 1, 1);
}

// ---------------------------------------------------------------------------
// Step 5 (L91-L93, Alg. 4).  bucket_q(f) = ((sigma_q f + nb/2) mod n) / nb
// is Alg. 4's range [ceil((J-1/2) nb), ceil((J+1/2) nb)).  A frequency with
// >= T of L_loc votes is selected in at least one of the first L_loc - T + 1
// location loops, so candidates f = a_{q0} p are enumerated only from those
// loops' preimage ranges; f is counted at the first such loop it is selected
// in (q < q0 bits must be clear) and then probed against the later loops'
// bitmaps, stopping once more than L_loc - T loops have missed.
// Dynamic smem: L_loc * B/32 u32 bitmaps.
// ---------------------------------------------------------------------------
struct VoteArgs {
  const uint8_t* records;
  RecLayout lay;
  const int* loc_slots;  // [L_loc] slot of each location loop, in vote order
  const uint32_t* loc_sigma;
  const uint32_t* loc_a;
  int Lloc, T, num, B, nb, log2nb, P;
  uint32_t nmask;
  int* hits;
  unsigned* hit_count;
  int max_hits;
};

__global__ void __launch_bounds__(256) k_vote(VoteArgs A) {
  extern __shared__ __align__(16) uint8_t smem[];
  uint32_t* bm = reinterpret_cast<uint32_t*>(smem);
  __shared__ uint32_t ssig[64];
  const int words = A.B >> 5;
  for (int q = 0; q < A.Lloc; ++q) {
    const uint32_t* src = reinterpret_cast<const uint32_t*>(A.records + (int64_t)A.loc_slots[q] * A.lay.rec_bytes +
                                                             A.lay.off_bitmap);
    for (int i = threadIdx.x; i < words; i += blockDim.x) bm[q * words + i] = src[i];
  }
  if (threadIdx.x < A.Lloc) ssig[threadIdx.x] = A.loc_sigma[threadIdx.x];
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int cpj = A.nb / A.P;  // chunks per bucket
  const int64_t per_q = (int64_t)A.num * cpj;
  const int64_t items = (int64_t)(A.Lloc - A.T + 1) * per_q;
  const uint32_t half = (uint32_t)(A.nb >> 1);
  // uniform trip count per warp so that ballots see every lane
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t start = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t warp_start = start - lane;
  for (int64_t it0 = warp_start; it0 < items; it0 += stride) {
    const int64_t it = it0 + lane;
    const bool valid_item = it < items;
    int q0 = 0;
    uint32_t a = 0, p = 0;
    if (valid_item) {
      q0 = (int)(it / per_q);
      const int64_t rem = it - (int64_t)q0 * per_q;
      const int jidx = (int)(rem / cpj);
      const int chunk = (int)(rem - (int64_t)jidx * cpj);
      const int* Jl = reinterpret_cast<const int*>(A.records + (int64_t)A.loc_slots[q0] * A.lay.rec_bytes +
                                                   A.lay.off_J);
      const uint32_t Jv = (uint32_t)Jl[jidx];
      p = (Jv * (uint32_t)A.nb - half + (uint32_t)(chunk * A.P)) & A.nmask;
      a = A.loc_a[q0];
    }
    for (int t = 0; t < A.P; ++t) {
      bool hit = false;
      uint32_t f = 0;
      if (valid_item) {
        f = (a * ((p + (uint32_t)t) & A.nmask)) & A.nmask;
        bool fresh = true;
        for (int q = 0; q < q0; ++q) {
          const uint32_t b = ((ssig[q] * f + half) & A.nmask) >> A.log2nb;
          if ((bm[q * words + (b >> 5)] >> (b & 31)) & 1u) {
            fresh = false;
            break;
          }
        }
        if (fresh) {
          const int allowed = A.Lloc - A.T - q0;
          int votes = 1, miss = 0;
          for (int q = q0 + 1; q < A.Lloc; ++q) {
            const uint32_t b = ((ssig[q] * f + half) & A.nmask) >> A.log2nb;
            if ((bm[q * words + (b >> 5)] >> (b & 31)) & 1u) {
              ++votes;
            } else if (++miss > allowed) {
              break;
            }
          }
          hit = votes >= A.T;
        }
      }
      const unsigned ball = __ballot_sync(kFull, hit);
      if (ball) {
        unsigned base = 0;
        if (lane == __ffs(ball) - 1) base = atomicAdd(A.hit_count, (unsigned)__popc(ball));
        base = __shfl_sync(kFull, base, __ffs(ball) - 1);
        if (hit) {
          const unsigned slot = base + __popc(ball & ((1u << lane) - 1));
          if ((int)slot < A.max_hits) A.hits[slot] = (int)f;
        }
      }
    }
  }
}

// ---------------------------------------------------------------------------
// Step 6 (L95, Alg. 5).  For hit f and every loop (slot) l:
//   p = sigma_l f mod n, h = p / nb, d = p mod nb; if d > nb/2: h = h+1 mod B, d -= nb;
//   v_l = u^_l[h] * e^{-2 pi i tau_l f / n} / G^(-d)
// then val = median(Re v) + i median(Im v), rank (L-1)/2 ascending.
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

__device__ __forceinline__ double rank_select(const double* v, int L, int med) {
  for (int i = 0; i < L; ++i) {
    int r = 0;
    for (int j = 0; j < L; ++j) r += (v[j] < v[i]) || (v[j] == v[i] && j < i);
    if (r == med) return v[i];
  }
  return v[0];
}

__global__ void __launch_bounds__(128) k_estimate(EstArgs A) {
  const int H = min((int)*A.hit_count, A.max_hits);
  double re[kMaxLoops], im[kMaxLoops];
  for (int h = blockIdx.x * blockDim.x + threadIdx.x; h < H; h += gridDim.x * blockDim.x) {
    const uint32_t f = (uint32_t)A.hits[h];
    for (int l = 0; l < A.L; ++l) {
      const SlotParam sp = A.slots[l];
      const uint32_t p = (sp.sigma * f) & A.nmask;
      int hb = (int)(p >> A.log2nb);
      int d = (int)(p & (uint32_t)(A.nb - 1));
      if (d > (A.nb >> 1)) {
        hb = (hb + 1) & (A.B - 1);
        d -= A.nb;
      }
      const double2 g = A.ghat[(A.nb >> 1) - d];  // G^(-d)
      const double2 b = reinterpret_cast<const double2*>(A.records + (int64_t)l * A.lay.rec_bytes)[hb];
      const uint32_t tph = (sp.tau * f) & A.nmask;
      double sn, cs;
      sincospi(2.0 * (double)tph / A.n, &sn, &cs);
      // b * e^{-i phi} with e^{-i phi} = cs - i sn
      const double zr = b.x * cs + b.y * sn;
      const double zi = b.y * cs - b.x * sn;
      // (zr + i zi) / (g.x + i g.y)
      const double den = g.x * g.x + g.y * g.y;
      re[l] = (zr * g.x + zi * g.y) / den;
      im[l] = (zi * g.x - zr * g.y) / den;
      if (A.per_loop) A.per_loop[(int64_t)h * A.L + l] = make_double2(re[l], im[l]);
    }
    const int med = (A.L - 1) >> 1;
    const double vr = rank_select(re, A.L, med);
    const double vi = rank_select(im, A.L, med);
    A.hit_vals[h] = make_double2(vr, vi);
    A.hit_keys[h] = (uint64_t)__double_as_longlong(__dadd_rn(__dmul_rn(vr, vr), __dmul_rn(vi, vi)));
  }
}

// ---------------------------------------------------------------------------
// Output: the k hits of largest |val|^2 (ties to the smaller f), written in
// ascending f; pads loc = -1, val = 0.  One CTA of 1024 threads.
// Dynamic smem: 4096 u32 hist + 64 ints + 2 * kp2 ints (sort buffer).
// ---------------------------------------------------------------------------
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
  int* sf = reinterpret_cast<int*>(smem + 4096 * 4 + 64 * 4);
  int* si = sf + kp2;
  const int H = min((int)*hit_count, max_hits);
  if (threadIdx.x == 0 && (int)*hit_count > max_hits) atomicOr(status, 1);
  const int K = min(k, H);
  Prefix96 p{0, 0, 0, 0};  // matches everything
  if (H > K) p = block_radix_select(HitSrc{hit_keys, hits}, H, K, hist, sm);
  if (threadIdx.x == 0) sm[40] = 0;
  for (int i = threadIdx.x; i < kp2; i += blockDim.x) {
    sf[i] = 0x7FFFFFFF;
    si[i] = -1;
  }
  __syncthreads();
  for (int i = threadIdx.x; i < H; i += blockDim.x) {
    if (ge96(p, hit_keys[i], ~(uint32_t)hits[i])) {
      const int pos = atomicAdd(&sm[40], 1);
      if (pos < kp2) {
        sf[pos] = hits[i];
        si[pos] = i;
      }
    }
  }
  __syncthreads();
  if (threadIdx.x == 0 && sm[40] != K) atomicOr(status + 2, 1);
  // bitonic sort of (sf, si) by sf ascending
  for (int size = 2; size <= kp2; size <<= 1) {
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
      for (int t = threadIdx.x; t < (kp2 >> 1); t += blockDim.x) {
        const int i = 2 * t - (t & (stride - 1));
        const int jn = i + stride;
        const bool up = (i & size) == 0;
        const int a = sf[i], b = sf[jn];
        if ((a > b) == up) {
          sf[i] = b;
          sf[jn] = a;
          const int ti = si[i];
          si[i] = si[jn];
          si[jn] = ti;
        }
      }
      __syncthreads();
    }
  }
  for (int j = threadIdx.x; j < k; j += blockDim.x) {
    if (j < K) {
      locs[j] = sf[j];
      vals[j] = hit_vals[si[j]];
    } else {
      locs[j] = -1;
      vals[j] = make_double2(0.0, 0.0);
    }
  }
}

}  // namespace cusfft
