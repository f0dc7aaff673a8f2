// fft.cuh — Step 3 (batched over loops as in L232): batched
// B-point forward FFT, fp64, in shared memory.  Replaces the paper's batched
// cuFFT call (north_star: no cuFFT on the hot path).
//
// B <= 2048: one pass, a CTA transforms 1024/B whole sequences.
// B  > 2048: four-step, B = B1 * B2:
//   pass 1: for each column c < B2, the B1-point FFT of u[c + B2 j1] (stride B2),
//           times e^{-2 pi i c k1 / B}, stored back at c + B2 k1;
//   pass 2: for each k1 < B1, the B2-point FFT of v[B2 k1 + c] (contiguous),
//           stored at u^[k1 + B1 k2].
// Inside a CTA: Stockham autosort (natural order in and out), radix-8 stages
// after one radix-2/4 stage when log2(M) is not a multiple of 3, with
// padded smem indexing pad(i) = i + i/8 + i/128 (conflict-free radix-8
// strides; the extra element per 128 skews consecutive 128-point sequences
// so that reading one element of each of them is not a bank conflict).
//
// Pass 2 (and the single pass) also produce the cutoff keys of the location
// loops: key = bits(re*re + im*im) (non-negative fp64 orders like its bit
// pattern) and a 4096-bin histogram of the key's top 12 bits below the sign
// (exponent + 1 mantissa bit), consumed by k_select.
#pragma once
#include "common.cuh"

namespace cusfft {

__device__ __forceinline__ int fft_pad(int i) { return i + (i >> 3) + (i >> 7); }
// elements of a padded workspace holding E
__host__ __device__ constexpr int fft_pad_n(int E) { return E + E / 8 + E / 128 + 1; }

__device__ __forceinline__ double2 cmul(double2 a, double2 b) {
  return make_double2(a.x * b.x - a.y * b.y, a.x * b.y + a.y * b.x);
}
__device__ __forceinline__ double2 cadd(double2 a, double2 b) { return make_double2(a.x + b.x, a.y + b.y); }
__device__ __forceinline__ double2 csub(double2 a, double2 b) { return make_double2(a.x - b.x, a.y - b.y); }
// multiply by -i
__device__ __forceinline__ double2 cmul_mi(double2 a) { return make_double2(a.y, -a.x); }

template <int R>
__device__ __forceinline__ void dft(double2* v);

template <>
__device__ __forceinline__ void dft<2>(double2* v) {
  double2 a = v[0], b = v[1];
  v[0] = cadd(a, b);
  v[1] = csub(a, b);
}

template <>
__device__ __forceinline__ void dft<4>(double2* v) {
  double2 s02 = cadd(v[0], v[2]), d02 = csub(v[0], v[2]);
  double2 s13 = cadd(v[1], v[3]), d13 = cmul_mi(csub(v[1], v[3]));
  v[0] = cadd(s02, s13);
  v[2] = csub(s02, s13);
  v[1] = cadd(d02, d13);
  v[3] = csub(d02, d13);
}

template <>
__device__ __forceinline__ void dft<8>(double2* v) {
  const double h = 0.70710678118654752440084436210485;  // 1/sqrt(2)
  double2 e[4] = {v[0], v[2], v[4], v[6]};
  double2 o[4] = {v[1], v[3], v[5], v[7]};
  dft<4>(e);
  dft<4>(o);
  // o[k] *= e^{-2 pi i k / 8}
  o[1] = make_double2(h * (o[1].x + o[1].y), h * (o[1].y - o[1].x));
  o[2] = cmul_mi(o[2]);
  o[3] = make_double2(h * (o[3].y - o[3].x), -h * (o[3].x + o[3].y));
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    v[k] = cadd(e[k], o[k]);
    v[k + 4] = csub(e[k], o[k]);
  }
}

// One Stockham stage of radix R over E elements (E/M sequences of length M) in
// S, jobs strided over NT threads.  Ns = product of the radices done so far.
template <int R, int M, int E, int NT, bool TWS = false>
__device__ __forceinline__ void stockham_stage(double2* S, int Ns, const double2* __restrict__ tw, int B) {
  constexpr int JOBS = E / R;
  constexpr int PER = (JOBS + NT - 1) / NT;
  constexpr int MR = M / R;
  double2 v[PER][R];
  int dst[PER];
  const int twstep = B / (Ns * R);
#pragma unroll
  for (int p = 0; p < PER; ++p) {
    const int job = threadIdx.x + p * NT;
    dst[p] = -1;
    if (job < JOBS) {
      const int sq = job / MR, j = job % MR;
      const int base = sq * M;
#pragma unroll
      for (int r = 0; r < R; ++r) v[p][r] = S[fft_pad(base + j + r * MR)];
      const int kk = j & (Ns - 1);
      if (Ns > 1) {
#pragma unroll
        for (int r = 1; r < R; ++r) v[p][r] = cmul(v[p][r], TWS ? tw[kk * r * twstep] : __ldg(tw + kk * r * twstep));
      }
      dft<R>(v[p]);
      dst[p] = base + (j - kk) * R + kk;
    }
  }
  __syncthreads();
#pragma unroll
  for (int p = 0; p < PER; ++p) {
    if (dst[p] >= 0) {
#pragma unroll
      for (int r = 0; r < R; ++r) S[fft_pad(dst[p] + r * Ns)] = v[p][r];
    }
  }
  __syncthreads();
}

// tw: table of e^{-2 pi i t / B}; TWS: tw lives in shared memory.
template <int M, int E, int NT, bool TWS = false>
__device__ __forceinline__ void fft_smem(double2* S, const double2* __restrict__ tw, int B) {
  constexpr int LOGM = (M >= 4096) ? 12 : (M >= 2048) ? 11 : (M >= 1024) ? 10 : (M >= 512) ? 9 : (M >= 256) ? 8
                       : (M >= 128) ? 7 : (M >= 64) ? 6 : (M >= 32) ? 5 : (M >= 16) ? 4 : (M >= 8) ? 3 : (M >= 4) ? 2 : 1;
  constexpr int REM = LOGM % 3;
  int Ns = 1;
  if constexpr (REM == 1) {
    stockham_stage<2, M, E, NT, TWS>(S, Ns, tw, B);
    Ns *= 2;
  } else if constexpr (REM == 2) {
    stockham_stage<4, M, E, NT, TWS>(S, Ns, tw, B);
    Ns *= 4;
  }
  if constexpr (LOGM >= 3) {
#pragma unroll 1
    for (int s = 0; s < LOGM / 3; ++s) {
      stockham_stage<8, M, E, NT, TWS>(S, Ns, tw, B);
      Ns *= 8;
    }
  }
}

struct FftPassArgs {
  const double2* in;
  double2* out;
  const double2* tw;
  int B;
  int log_seq_per_slot;  // sequences per slot = 2^log_seq_per_slot
  int total_seq;
  int64_t in_ls, out_ls;  // slot strides (elements)
  int in_cs, in_es, out_cs, out_es;
  int twiddle;  // pass 1: multiply element e of column col by tw[col*e mod B]
  // cutoff keys (pass 2 / single pass only): slot -> location index or -1
  const int* key_index;   // [slots of this rank], may be null
  uint64_t* keys;         // [n_sel][B]
  uint32_t* hist;         // [n_sel][4096] top-digit histograms (null: none)
};

// E = elements per CTA, NT = threads per CTA.  Dynamic smem: fft_smem_bytes(E).
__host__ __device__ constexpr int fft_smem_bytes(int E) { return fft_pad_n(E) * 16 + 4096 * 4 + E * 16; }

template <int M, int E, int NT>
__global__ void __launch_bounds__(NT) k_fft(FftPassArgs A) {
  pdl_wait();
  KTRACE(A.twiddle ? 5 : 6);
  constexpr int NSEQ = E / M;
  extern __shared__ __align__(16) uint8_t fsm[];
  double2* S = reinterpret_cast<double2*>(fsm);
  uint32_t* shist = reinterpret_cast<uint32_t*>(fsm + fft_pad_n(E) * sizeof(double2));
  double2* twl = reinterpret_cast<double2*>(fsm + fft_pad_n(E) * sizeof(double2) + 4096 * 4);  // omega_M^t, t < M
  const int q0 = blockIdx.x * NSEQ;
  for (int t = threadIdx.x; t < M; t += NT) twl[t] = __ldg(A.tw + (int64_t)t * (A.B / M));
  if (blockIdx.x == 0) TRACE(A.twiddle ? 2 : 4);
  const bool col_fast_in = (A.in_cs == 1);
  const int spm = (1 << A.log_seq_per_slot) - 1;
  {  // all E/NT loads of a thread in flight before the first smem store
    constexpr int PER = E / NT;
    double2 buf[PER];
    int dst[PER];
#pragma unroll
    for (int u = 0; u < PER; ++u) {
      const int t = threadIdx.x + u * NT;
      int sq, e;
      if (col_fast_in) {
        sq = t % NSEQ;
        e = t / NSEQ;
      } else {
        sq = t / M;
        e = t % M;
      }
      const int q = q0 + sq;
      dst[u] = -1;
      if (q < A.total_seq) {
        const int l = q >> A.log_seq_per_slot, col = q & spm;
        buf[u] = __ldg(A.in + (int64_t)l * A.in_ls + (int64_t)col * A.in_cs + (int64_t)e * A.in_es);
        dst[u] = fft_pad(sq * M + e);
      }
    }
#pragma unroll
    for (int u = 0; u < PER; ++u)
      if (dst[u] >= 0) S[dst[u]] = buf[u];
  }
  __syncthreads();
  fft_smem<M, E, NT, true>(S, twl, M);
  // keys: a CTA's sequences all belong to one slot when NSEQ <= seq_per_slot
  const bool one_slot = NSEQ <= (1 << A.log_seq_per_slot);
  int kidx = -1;
  if (A.key_index && one_slot) kidx = A.key_index[q0 >> A.log_seq_per_slot];
  const bool hist = A.hist != nullptr;
  if (kidx >= 0 && hist) {
    for (int i = threadIdx.x; i < 4096; i += NT) shist[i] = 0;
    __syncthreads();
  }
  const bool col_fast_out = (A.out_cs == 1);
  for (int t = threadIdx.x; t < E; t += NT) {
    int sq, e;
    if (col_fast_out) {
      sq = t % NSEQ;
      e = t / NSEQ;
    } else {
      sq = t / M;
      e = t % M;
    }
    const int q = q0 + sq;
    if (q < A.total_seq) {
      const int l = q >> A.log_seq_per_slot, col = q & spm;
      double2 v = S[fft_pad(sq * M + e)];
      if (A.twiddle) v = cmul(v, __ldg(A.tw + (((int64_t)col * e) & (A.B - 1))));
      const int64_t opos = (int64_t)col * A.out_cs + (int64_t)e * A.out_es;
      A.out[(int64_t)l * A.out_ls + opos] = v;
      if (A.key_index) {
        const int ki = one_slot ? kidx : A.key_index[l];
        if (ki >= 0) {
          const uint64_t key =
              (uint64_t)__double_as_longlong(__dadd_rn(__dmul_rn(v.x, v.x), __dmul_rn(v.y, v.y)));
          A.keys[(int64_t)ki * A.B + opos] = key;
          const uint32_t d = (uint32_t)(key >> 51) & 0xFFFu;
          if (!hist) {
          } else if (one_slot) {
            atomicAdd(&shist[d], 1u);
          } else {
            atomicAdd(&A.hist[(int64_t)ki * 4096 + d], 1u);
          }
        }
      }
    }
  }
  if (kidx >= 0 && hist) {
    __syncthreads();
    for (int i = threadIdx.x; i < 4096; i += NT)
      if (shist[i]) atomicAdd(&A.hist[(int64_t)kidx * 4096 + i], shist[i]);
  }
  if (A.twiddle) TRACE_END(3); else TRACE_END(5);
}

}  // namespace cusfft
