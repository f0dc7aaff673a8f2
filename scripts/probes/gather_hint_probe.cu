// Phase-1 read-pattern probe: address-sorted 16-B gathers (2.8 M from 256 MiB,
// as in C3's fold phase 1) scattered into a 45 MB staging buffer kept in the
// persisting set-aside.  Varies the L2 fetch-size hint of the x loads and the
// loads in flight per thread.  Prints event times (mean of 8 after 2 warm-ups,
// bench.py's L2 flush before each).
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
#include <algorithm>
#include <cuda_runtime.h>

template <int H, int U>
__global__ void __launch_bounds__(256) gather(const double2* __restrict__ x, const uint32_t* __restrict__ pos,
                                              const uint32_t* __restrict__ dst, double2* S, int N) {
  uint64_t pf, pl;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pf));
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pl));
  const int T = gridDim.x * blockDim.x;
  for (int q0 = blockIdx.x * blockDim.x + threadIdx.x; q0 < N; q0 += U * T) {
    double2 v[U];
#pragma unroll
    for (int c = 0; c < U; ++c) {
      const int q = q0 + c * T;
      if (q < N) {
        const double2* p = x + pos[q];
        if (H == 64)
          asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.L2::64B.v2.f64 {%0, %1}, [%2], %3;"
                       : "=d"(v[c].x), "=d"(v[c].y) : "l"(p), "l"(pf));
        else if (H == 128)
          asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.L2::128B.v2.f64 {%0, %1}, [%2], %3;"
                       : "=d"(v[c].x), "=d"(v[c].y) : "l"(p), "l"(pf));
        else if (H == 256)
          asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.L2::256B.v2.f64 {%0, %1}, [%2], %3;"
                       : "=d"(v[c].x), "=d"(v[c].y) : "l"(p), "l"(pf));
        else
          asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f64 {%0, %1}, [%2], %3;"
                       : "=d"(v[c].x), "=d"(v[c].y) : "l"(p), "l"(pf));
      }
    }
#pragma unroll
    for (int c = 0; c < U; ++c) {
      const int q = q0 + c * T;
      if (q < N)
        asm volatile("st.global.L2::cache_hint.v2.f64 [%0], {%1, %2}, %3;" ::"l"(S + dst[q]), "d"(v[c].x),
                     "d"(v[c].y), "l"(pl));
    }
  }
}

__global__ void flush_read(const int4* __restrict__ p, size_t n, int* out) {
  int a = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    a ^= p[i].x ^ p[i].w;
  if (a == 12345) out[0] = a;
}

int main() {
  const uint32_t n = 1u << 24;
  const int N = 2800000;
  std::mt19937_64 rng(1);
  std::vector<uint32_t> pos(N), dst(N);
  for (auto& p : pos) p = (uint32_t)(rng() % n);
  std::sort(pos.begin(), pos.end());
  for (int i = 0; i < N; ++i) dst[i] = i;
  std::shuffle(dst.begin(), dst.end(), rng);
  double2 *x, *S;
  uint32_t *dpos, *ddst;
  uint8_t* fw;
  void* fr;
  int* fo;
  const size_t fb = 256ull << 20;
  cudaMalloc(&x, (size_t)n * 16);
  cudaMalloc(&S, (size_t)N * 16);
  cudaMalloc(&dpos, N * 4);
  cudaMalloc(&ddst, N * 4);
  cudaMalloc(&fw, fb);
  cudaMalloc(&fr, fb);
  cudaMalloc(&fo, 64);
  cudaMemset(x, 1, (size_t)n * 16);
  cudaMemset(fr, 1, fb);
  cudaMemcpy(dpos, pos.data(), N * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(ddst, dst.data(), N * 4, cudaMemcpyHostToDevice);
  cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)N * 16);
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  auto run = [&](const char* name, auto kern, int cps) {
    float tot = 0;
    for (int r = 0; r < 10; ++r) {
      cudaMemsetAsync(fw, 0, fb);
      flush_read<<<sms * 8, 256>>>((const int4*)fr, fb / 16, fo);
      cudaEventRecord(a);
      kern<<<sms * cps, 256>>>(x, dpos, ddst, S, N);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (r >= 2) tot += ms;
    }
    printf("%-28s cps %d: %.1f us\n", name, cps, 1e3 * tot / 8);
  };
  for (int cps : {4, 8}) {
    run("L2::64B  x8 in flight", gather<64, 8>, cps);
    run("L2::128B x8 in flight", gather<128, 8>, cps);
    run("L2::256B x8 in flight", gather<256, 8>, cps);
    run("no size hint x8", gather<0, 8>, cps);
    run("L2::64B  x16 in flight", gather<64, 16>, cps);
    run("L2::128B x16 in flight", gather<128, 16>, cps);
    run("L2::64B  x4 in flight", gather<64, 4>, cps);
  }
  printf("status %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
