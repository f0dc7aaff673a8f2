// plan_kernels.cuh — plan-time device kernels (not on the timed path):
// filter construction (DESIGN.md §3 [Z1]), its frequency
// response G^(q) (Alg. 5's filter_freq, L325) and the B-point twiddles (L87).
// Everything in fp64 with exact integer phase reduction before sincospi.
#pragma once
#include "common.cuh"

namespace cusfft {

// tw[t] = e^{-2 pi i t / B}, t in [0, B).
__global__ void k_twiddles(double2* tw, int B) {
  int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t < B) {
    double s, c;
    sincospi(2.0 * (double)t / (double)B, &s, &c);
    tw[t] = make_double2(c, -s);
  }
}

// Chebyshev polynomial T_m(y) for real y.
__device__ __forceinline__ double cheb_T(double m, double y) {
  if (fabs(y) <= 1.0) return cos(m * acos(y));
  if (y > 1.0) return cosh(m * acosh(y));
  // m = w - 1 is even for odd w, so T_m(-y) = T_m(y)
  return cosh(m * acosh(-y));
}

// Dolph-Chebyshev spectrum samples p_j = T_{w-1}(x0 cos(pi j / w)), j in [0, c].
__global__ void k_cheb_samples(double* pj, int w, double x0) {
  int j = blockIdx.x * blockDim.x + threadIdx.x;
  int c = (w - 1) / 2;
  if (j <= c) pj[j] = cheb_T((double)(w - 1), x0 * cospi((double)j / (double)w));
}

// Dolph-Chebyshev window (unnormalised) W(t) = p_0 + 2 sum_{j=1}^{c} p_j cos(2 pi j t / w)
// for t in [0, c] (the window is even; p_j = p_{w-j}).  One CTA per t; the phase
// index (j t) mod w is carried exactly in integers.
__global__ void __launch_bounds__(256) k_dc_window(const double* __restrict__ pj, double* win, int w) {
  __shared__ double red[8];
  const int t = blockIdx.x;
  const int c = (w - 1) / 2;
  const int64_t step = ((int64_t)blockDim.x * t) % w;
  int64_t m = ((int64_t)(threadIdx.x + 1) * t) % w;
  double acc = 0.0;
  for (int j = threadIdx.x + 1; j <= c; j += blockDim.x) {
    acc = fma(pj[j], cospi(2.0 * (double)m / (double)w), acc);
    m += step;
    if (m >= w) m -= w;
  }
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(kFull, acc, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0.0;
    for (int i = 0; i < (int)(blockDim.x >> 5); ++i) s += red[i];
    win[t] = pj[0] + 2.0 * s;
  }
}

// Gaussian window W(t) = exp(-t^2 / (2 s^2)), t in [0, c].
__global__ void k_gauss_window(double* win, int w, double s) {
  int t = blockIdx.x * blockDim.x + threadIdx.x;
  int c = (w - 1) / 2;
  if (t <= c) win[t] = exp(-((double)t * (double)t) / (2.0 * s * s));
}

// Unnormalised taps g_i = W(|i-c|) D(i-c), D(t) = sin(pi b t / n) / sin(pi t / n),
// D(0) = b; zero for w <= i < padded.
__global__ void k_taps(const double* __restrict__ win, double* taps, int w, int padded, int64_t n, int64_t b) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= padded) return;
  if (i >= w) {
    taps[i] = 0.0;
    return;
  }
  int c = (w - 1) / 2;
  int64_t t = i >= c ? (int64_t)(i - c) : (int64_t)(c - i);
  double D;
  if (t == 0) {
    D = (double)b;
  } else {
    int64_t num = (b * t) % (2 * n);  // sin(pi x) has period 2 in x
    D = sinpi((double)num / (double)n) / sinpi((double)t / (double)n);
  }
  taps[i] = win[t] * D;
}

// Single-CTA deterministic sum of taps[0..w) and scale so that the sum is 1.
__global__ void __launch_bounds__(1024) k_normalize(double* taps, int w) {
  __shared__ double red[32];
  __shared__ double total;
  double acc = 0.0;
  for (int i = threadIdx.x; i < w; i += blockDim.x) acc += taps[i];
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(kFull, acc, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0.0;
    for (int i = 0; i < (int)(blockDim.x >> 5); ++i) s += red[i];
    total = s;
  }
  __syncthreads();
  const double inv = 1.0 / total;
  for (int i = threadIdx.x; i < w; i += blockDim.x) taps[i] *= inv;
}

// G^(q) = sum_{i<w} g_i e^{-2 pi i q i / n} for q = -nb/2 .. nb/2, entry q + nb/2.
// One CTA per q; the phase index (q i) mod n is exact (n divides 2^64).
__global__ void __launch_bounds__(256) k_ghat(const double* __restrict__ taps, double2* ghat, int w, int64_t n, int nb) {
  __shared__ double rr[8], ri[8];
  const int64_t q = (int64_t)blockIdx.x - nb / 2;
  const uint64_t nmask = (uint64_t)n - 1;
  const uint64_t qm = (uint64_t)q & nmask;
  const uint64_t step = (qm * blockDim.x) & nmask;
  uint64_t m = (qm * threadIdx.x) & nmask;
  double re = 0.0, im = 0.0;
  for (int i = threadIdx.x; i < w; i += blockDim.x) {
    double s, c;
    sincospi(2.0 * (double)m / (double)n, &s, &c);
    re = fma(taps[i], c, re);
    im = fma(-taps[i], s, im);
    m = (m + step) & nmask;
  }
  for (int o = 16; o > 0; o >>= 1) {
    re += __shfl_xor_sync(kFull, re, o);
    im += __shfl_xor_sync(kFull, im, o);
  }
  if ((threadIdx.x & 31) == 0) {
    rr[threadIdx.x >> 5] = re;
    ri[threadIdx.x >> 5] = im;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    double a = 0.0, b = 0.0;
    for (int i = 0; i < (int)(blockDim.x >> 5); ++i) {
      a += rr[i];
      b += ri[i];
    }
    ghat[blockIdx.x] = make_double2(a, b);
  }
}

// Estimation tables (Alg. 5's filter_freq division and the phase of Def. 1):
// ginv[q] = 1 / G^(q) (complex reciprocal, q = -nb/2 .. nb/2, entry q + nb/2).
__global__ void k_ginv(const double2* __restrict__ ghat, double2* ginv, int m) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < m) {
    const double2 g = ghat[i];
    const double den = g.x * g.x + g.y * g.y;
    ginv[i] = make_double2(g.x / den, -g.y / den);
  }
}

// e^{-2 pi i m / n} for m = j << shift, j < count (the exact fraction m / n
// = j / 2^(log2n - shift) handed to sincospi).
__global__ void k_phase_table(double2* tab, int count, int shift, int log2n) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j < count) {
    double s, c;
    sincospi(2.0 * ldexp((double)j, shift - log2n), &s, &c);
    tab[j] = make_double2(c, -s);
  }
}

}  // namespace cusfft
