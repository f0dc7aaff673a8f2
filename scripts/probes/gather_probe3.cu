// Two-phase fold probe: (1) address-sorted gather of x, scatter 16-B values to
// an L2-resident staging buffer in (loop, tap) order; (2) ordered fold read.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>
constexpr int R = 13, B = 16384, L = 16;
__device__ __forceinline__ uint64_t pol_first() { uint64_t p; asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p)); return p; }
__device__ __forceinline__ uint64_t pol_last() { uint64_t p; asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p)); return p; }
template <int H>
__device__ __forceinline__ double2 ldx(const double2* p, uint64_t pol) {
  double2 v;
  if (H == 0) asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  if (H == 1) asm volatile("ld.global.nc.L1::no_allocate.L2::64B.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  if (H == 2) asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.L2::64B.v2.f64 {%0,%1}, [%2], %3;" : "=d"(v.x), "=d"(v.y) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ uint32_t pos_of(uint32_t d, uint32_t nmask) {
  uint32_t y = d / (R * B), rem = d % (R * B);
  uint32_t sigma = (0x9E3779B1u | 1u) + y * 2654435761u * 2u, tau = y * 7919u;
  return (sigma * rem + tau) & nmask;
}
template <int H, int ST>
__global__ void __launch_bounds__(256) phase1(const double2* __restrict__ x, const uint32_t* __restrict__ dst, double2* stage, int total, uint32_t nmask) {
  int t = blockIdx.x * blockDim.x + threadIdx.x, T = gridDim.x * blockDim.x;
  uint64_t pf = pol_first(), pl = pol_last();
  double2 v[8]; uint32_t d[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) {
    int q = t + c * T;
    d[c] = q < total ? __ldg(dst + q) : 0xFFFFFFFFu;
    v[c] = q < total ? ldx<H>(x + pos_of(d[c], nmask), pf) : make_double2(0, 0);
  }
#pragma unroll
  for (int c = 0; c < 8; ++c) if (d[c] != 0xFFFFFFFFu) {
    if (ST == 0) stage[d[c]] = v[c];
    else asm volatile("st.global.L2::cache_hint.v2.f64 [%0], {%1,%2}, %3;" :: "l"(stage + d[c]), "d"(v[c].x), "d"(v[c].y), "l"(pl));
  }
}
__global__ void __launch_bounds__(256) phase2(const double2* __restrict__ stage, const double* __restrict__ taps, double2* u) {
  int j = blockIdx.x * blockDim.x + threadIdx.x, y = blockIdx.y;
  double ar = 0, ai = 0;
  double2 v[R];
#pragma unroll
  for (int c = 0; c < R; ++c) v[c] = stage[(size_t)y * R * B + c * B + j];
#pragma unroll
  for (int c = 0; c < R; ++c) { double g = taps[c * B + j]; ar = __dadd_rn(ar, __dmul_rn(g, v[c].x)); ai = __dadd_rn(ai, __dmul_rn(g, v[c].y)); }
  u[(size_t)y * B + j] = make_double2(ar, ai);
}
int main() {
  size_t n = 1u << 24; uint32_t nmask = n - 1;
  double2 *x, *stage, *u; double* taps; char* flush; uint32_t* dst;
  cudaMalloc(&x, n * 16); cudaMalloc(&stage, (size_t)L * R * B * 16); cudaMalloc(&u, L * B * 16);
  cudaMalloc(&taps, R * B * 8); cudaMalloc(&flush, 512u << 20);
  cudaMemset(x, 0, n * 16); cudaMemset(taps, 0, R * B * 8);
  std::vector<std::pair<uint32_t, uint32_t>> e;
  for (uint32_t y = 0; y < L; ++y) for (uint32_t i = 0; i < R * B; ++i) {
    uint32_t d = y * R * B + i;
    uint32_t sigma = (0x9E3779B1u | 1u) + y * 2654435761u * 2u, tau = y * 7919u;
    e.push_back({(sigma * i + tau) & nmask, d});
  }
  std::sort(e.begin(), e.end());
  std::vector<uint32_t> h(e.size()); for (size_t i = 0; i < e.size(); ++i) h[i] = e[i].second;
  int total = h.size();
  cudaMalloc(&dst, total * 4); cudaMemcpy(dst, h.data(), total * 4, cudaMemcpyHostToDevice);
  cudaEvent_t a, b, c2; cudaEventCreate(&a); cudaEventCreate(&b); cudaEventCreate(&c2);
  int T = (total + 7) / 8;
  auto run = [&](int variant) {
    float b1 = 1e9, b2 = 1e9;
    for (int it = 0; it < 6; ++it) {
      cudaMemset(flush, it, 512u << 20);
      cudaEventRecord(a);
      if (variant == 0) phase1<0, 0><<<(T + 255) / 256, 256>>>(x, dst, stage, total, nmask);
      if (variant == 1) phase1<1, 0><<<(T + 255) / 256, 256>>>(x, dst, stage, total, nmask);
      if (variant == 2) phase1<2, 1><<<(T + 255) / 256, 256>>>(x, dst, stage, total, nmask);
      cudaEventRecord(b);
      phase2<<<dim3(B / 256, L), 256>>>(stage, taps, u);
      cudaEventRecord(c2); cudaEventSynchronize(c2);
      float t1, t2; cudaEventElapsedTime(&t1, a, b); cudaEventElapsedTime(&t2, b, c2);
      if (it > 0) { b1 = std::min(b1, t1); b2 = std::min(b2, t2); }
    }
    printf("variant %d: phase1 %.2f us phase2 %.2f us\n", variant, b1 * 1e3, b2 * 1e3);
  };
  run(0); run(1); run(2);
  return 0;
}
