// Fold gather issue-order probe (C3 shape: n 2^24, L 16, B 16384, w 175347).
// Does issuing each CTA's gathers in address order (so that all resident CTAs
// sweep x together) beat the random-order direct gather without a global
// staging buffer?  Variants:
//   direct      thread per (slot, bucket), its R rounds' gathers in flight
//   band<D>     CTA of 256 buckets; its R*256 samples sorted by address at plan
//               time (uint16 smem slot codes); D sorted loads per thread in
//               flight, each stored to smem, then the fold from smem
//   stage       global address-sorted gather into a staging buffer (phase 1 only)
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <random>
#include <vector>
#include <cuda_runtime.h>

constexpr int B = 16384, L = 16, NT = 256;
__device__ __forceinline__ double2 ldg64(const double2* p) {
  double2 v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::64B.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  return v;
}
__device__ __forceinline__ double2 ldg(const double2* p) {
  double2 v;
  asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  return v;
}
struct Sl { uint32_t sigma, tau; };

template <int R>
__global__ void __launch_bounds__(256) direct(const double2* __restrict__ x, const double* __restrict__ taps,
                                              const Sl* sl, double2* u, int w, uint32_t nmask) {
  int j = blockIdx.x * 256 + threadIdx.x, s = blockIdx.y;
  uint32_t sg = sl[s].sigma, tu = sl[s].tau;
  double2 v[R];
#pragma unroll
  for (int c = 0; c < R; ++c) {
    int i = j + c * B;
    if (i < w) v[c] = ldg64(x + ((sg * (uint32_t)i + tu) & nmask));
  }
  double ar = 0, ai = 0;
#pragma unroll
  for (int c = 0; c < R; ++c) {
    int i = j + c * B;
    if (i < w) { double g = __ldg(taps + i); ar = __dadd_rn(ar, __dmul_rn(g, v[c].x)); ai = __dadd_rn(ai, __dmul_rn(g, v[c].y)); }
  }
  u[(size_t)s * B + j] = make_double2(ar, ai);
}

// codes: [grid][R*256] uint16, smem slot rr*256+tl in address order, 0xFFFF = none
template <int R, int D, bool HINT>
__global__ void __launch_bounds__(256, 4) band(const double2* __restrict__ x, const double* __restrict__ taps,
                                               const Sl* sl, const uint16_t* __restrict__ codes, double2* u, int w,
                                               uint32_t nmask) {
  __shared__ double2 S[R * NT];
  const int t = threadIdx.x;
  const int b = blockIdx.x;
  const int s = b / (B / NT), j0 = (b % (B / NT)) * NT;
  const uint32_t sg = sl[s].sigma, tu = sl[s].tau;
  const uint16_t* cp = codes + (size_t)b * R * NT + t;
#pragma unroll
  for (int c0 = 0; c0 < R; c0 += D) {
    double2 v[D];
    uint16_t cd[D];
#pragma unroll
    for (int d = 0; d < D; ++d) {
      if (c0 + d < R) {
        cd[d] = __ldcs(cp + (c0 + d) * NT);
        if (cd[d] != 0xFFFF) {
          int i = j0 + (cd[d] & 255) + (cd[d] >> 8) * B;
          const double2* p = x + ((sg * (uint32_t)i + tu) & nmask);
          v[d] = HINT ? ldg64(p) : ldg(p);
        }
      }
    }
#pragma unroll
    for (int d = 0; d < D; ++d)
      if (c0 + d < R && cd[d] != 0xFFFF) S[cd[d]] = v[d];
  }
  __syncthreads();
  double ar = 0, ai = 0;
#pragma unroll
  for (int rr = 0; rr < R; ++rr) {
    int i = j0 + t + rr * B;
    if (i < w) { double g = __ldg(taps + i); double2 q = S[rr * NT + t]; ar = __dadd_rn(ar, __dmul_rn(g, q.x)); ai = __dadd_rn(ai, __dmul_rn(g, q.y)); }
  }
  u[(size_t)s * B + j0 + t] = make_double2(ar, ai);
}

template <bool HINT>
__global__ void __launch_bounds__(256) stage(const double2* __restrict__ x, const uint32_t* __restrict__ spos,
                                             double2* st, int total) {
  const int T = gridDim.x * blockDim.x;
  for (int q0 = blockIdx.x * blockDim.x + threadIdx.x; q0 < total; q0 += 8 * T) {
    double2 v[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) if (q0 + c * T < total) v[c] = HINT ? ldg64(x + __ldg(spos + q0 + c * T)) : ldg(x + __ldg(spos + q0 + c * T));
#pragma unroll
    for (int c = 0; c < 8; ++c) if (q0 + c * T < total) __stcg(st + q0 + c * T, v[c]);
  }
}


// Persistent sweep: one CTA per SM holds up to 4 tiles (256 buckets x R rounds
// of one slot) in shared memory; the CTA's samples sorted by address (uint16
// smem-slot codes), K loads in flight per thread; then the fold from smem.
template <int R, int K>
__global__ void __launch_bounds__(1024, 1) persist(const double2* __restrict__ x, const double* __restrict__ taps,
                                                   const Sl* sl, const uint16_t* __restrict__ codes,
                                                   const int* __restrict__ offs, const int2* __restrict__ tiles,
                                                   int tile0, int ntiles, double2* u, int w, uint32_t nmask) {
  extern __shared__ double2 SM[];
  __shared__ uint32_t tsig[4], ttau[4];
  __shared__ int tj0[4], tsl[4];
  const int t = threadIdx.x, c = blockIdx.x, G = gridDim.x;
  const int a0 = tile0 + (int)((long long)c * ntiles / G), a1 = tile0 + (int)((long long)(c + 1) * ntiles / G);
  if (t < 4 && a0 + t < a1) {
    int2 tl = tiles[a0 + t];
    tsl[t] = tl.x; tj0[t] = tl.y; tsig[t] = sl[tl.x].sigma; ttau[t] = sl[tl.x].tau;
  }
  __syncthreads();
  const int e0 = offs[c], e1 = offs[c + 1];
  uint16_t* scode = reinterpret_cast<uint16_t*>(SM + 4 * R * 256);
  for (int e = t; e < e1 - e0; e += 1024) scode[e] = __ldcs(codes + e0 + e);
  __syncthreads();
  const int ne = e1 - e0;
  for (int e = t; e < ne; e += 1024 * K) {
    uint16_t cd[K];
    double2 v[K];
#pragma unroll
    for (int d = 0; d < K; ++d) {
      const int ee = e + d * 1024;
      if (ee < ne) {
        cd[d] = scode[ee];
        const int lt = cd[d] / (R * 256), rem = cd[d] - lt * (R * 256);
        const int rr = rem >> 8, tl = rem & 255;
        const uint32_t i = (uint32_t)(tj0[lt] + tl + rr * B);
        v[d] = ldg64(x + ((tsig[lt] * i + ttau[lt]) & nmask));
      }
    }
#pragma unroll
    for (int d = 0; d < K; ++d)
      if (e + d * 1024 < ne) SM[cd[d]] = v[d];
  }
  __syncthreads();
  const int lt = t >> 8, tl = t & 255;
  if (a0 + lt < a1) {
    double ar = 0, ai = 0;
#pragma unroll
    for (int rr = 0; rr < R; ++rr) {
      int i = tj0[lt] + tl + rr * B;
      if (i < w) { double g = __ldg(taps + i); double2 q = SM[lt * R * 256 + rr * 256 + tl]; ar = __dadd_rn(ar, __dmul_rn(g, q.x)); ai = __dadd_rn(ai, __dmul_rn(g, q.y)); }
    }
    u[(size_t)tsl[lt] * B + tj0[lt] + tl] = make_double2(ar, ai);
  }
}

__global__ void readall(const int4* __restrict__ p, size_t n, int* out) {
  int acc = 0;
  for (size_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) { int4 v = __ldcs(p + i); acc ^= v.x ^ v.w; }
  if (acc == 0x7fffffff) out[0] = acc;
}
int main(int argc, char** argv) {
  const double tol = argc > 1 ? atof(argv[1]) : 1e-7;
  const uint32_t n = 1u << 24, nmask = n - 1;
  int w = (int)(acosh(1.0 / tol) / (M_PI * 0.5 / B));
  if (w % 2 == 0) --w;
  constexpr int R = 11;
  if ((w + B - 1) / B != R) { printf("R mismatch %d\n", (w + B - 1) / B); return 1; }
  printf("w=%d R=%d L=%d\n", w, R, L);
  std::mt19937_64 rng(3);
  std::vector<Sl> sl(L);
  for (auto& q : sl) { q.sigma = (uint32_t)(rng() & nmask) | 1u; q.tau = (uint32_t)(rng() & nmask); }
  double2 *x, *u, *st; double* taps; Sl* dsl; uint16_t* dcodes; uint32_t* dspos;
  char* fw; int* fr;
  cudaMalloc(&x, (size_t)n * 16); cudaMalloc(&u, (size_t)L * B * 16); cudaMalloc(&taps, (size_t)R * B * 8);
  cudaMalloc(&st, (size_t)L * w * 16); cudaMalloc(&dsl, L * sizeof(Sl));
  cudaMalloc(&fw, 256u << 20); cudaMalloc(&fr, 256u << 20);
  cudaMemset(x, 0, (size_t)n * 16); cudaMemset(taps, 0, (size_t)R * B * 8); cudaMemset(fr, 0, 256u << 20);
  cudaMemcpy(dsl, sl.data(), L * sizeof(Sl), cudaMemcpyHostToDevice);
  const int grid = L * (B / NT);
  std::vector<uint16_t> codes((size_t)grid * R * NT, 0xFFFF);
  for (int b = 0; b < grid; ++b) {
    int s = b / (B / NT), j0 = (b % (B / NT)) * NT;
    std::vector<std::pair<uint32_t, uint16_t>> e;
    for (int rr = 0; rr < R; ++rr)
      for (int tl = 0; tl < NT; ++tl) {
        int i = j0 + tl + rr * B;
        if (i < w) e.push_back({(sl[s].sigma * (uint32_t)i + sl[s].tau) & nmask, (uint16_t)(rr * NT + tl)});
      }
    std::sort(e.begin(), e.end());
    for (size_t q = 0; q < e.size(); ++q) codes[(size_t)b * R * NT + q] = e[q].second;
  }
  cudaMalloc(&dcodes, codes.size() * 2);
  cudaMemcpy(dcodes, codes.data(), codes.size() * 2, cudaMemcpyHostToDevice);
  std::vector<uint32_t> spos;
  for (int s = 0; s < L; ++s) for (int i = 0; i < w; ++i) spos.push_back((sl[s].sigma * (uint32_t)i + sl[s].tau) & nmask);
  std::sort(spos.begin(), spos.end());
  cudaMalloc(&dspos, spos.size() * 4);
  cudaMemcpy(dspos, spos.data(), spos.size() * 4, cudaMemcpyHostToDevice);
  const int total = (int)spos.size();
  cudaEvent_t a, bb; cudaEventCreate(&a); cudaEventCreate(&bb);
  auto timeit = [&](const char* name, auto launch) {
    float sum = 0; int reps = 20;
    for (int r = 0; r < reps + 3; ++r) {
      cudaMemsetAsync(fw, r, 256u << 20); readall<<<148 * 8, 256>>>((const int4*)fr, (256u << 20) / 16, (int*)u);
      cudaEventRecord(a); launch(); cudaEventRecord(bb); cudaEventSynchronize(bb);
      float ms; cudaEventElapsedTime(&ms, a, bb);
      if (r >= 3) sum += ms;
    }
    cudaError_t e = cudaGetLastError();
    printf("%-14s %8.2f us  (%.1f G samples/s) %s\n", name, 1e3 * sum / reps, (double)L * w / (sum / reps * 1e-3) / 1e9,
           e ? cudaGetErrorString(e) : "");
  };


  // banded stage orders: key = (pos >> bsh, destination tile, pos)
  for (int bands : {1, 16, 64, 256, 1024}) {
    int bsh = 24 - __builtin_ctz(bands);
    std::vector<std::pair<uint64_t, uint32_t>> e;
    e.reserve((size_t)L * w);
    for (int s = 0; s < L; ++s) for (int i2 = 0; i2 < w; ++i2) {
      uint32_t pos = (sl[s].sigma * (uint32_t)i2 + sl[s].tau) & nmask;
      uint32_t tile = (uint32_t)(s * (B / 256) + (i2 % B) / 256);
      uint64_t key = bands == 1 ? pos : (((uint64_t)(pos >> bsh) << 44) | ((uint64_t)tile << 24) | pos);
      e.push_back({key, pos});
    }
    std::sort(e.begin(), e.end());
    std::vector<uint32_t> sp2(e.size());
    for (size_t q = 0; q < e.size(); ++q) sp2[q] = e[q].second;
    cudaMemcpy(dspos, sp2.data(), sp2.size() * 4, cudaMemcpyHostToDevice);
    char nm[64]; snprintf(nm, sizeof nm, "stage bands=%d", bands);
    timeit(nm, [&] { stage<true><<<148 * 8, 256>>>(x, dspos, st, total); });
  }
  timeit("stage", [&] { stage<true><<<148 * 8, 256>>>(x, dspos, st, total); });
  timeit("direct", [&] { direct<R><<<dim3(B / 256, L), 256>>>(x, taps, dsl, u, w, nmask); });
  return 0;
}
