// Staging write-back probe (DESIGN.md §6.2 "The staging writes reach DRAM").
// Mimics fold phase 1: address-sorted 16-B gathers from a 256 MiB x, each
// sample scattered to a random slot of a 45 MB staging buffer held in the
// persisting L2 set-aside; then a coalesced read of the staging (phase 2
// analogue).  Variants isolate why ~35 MB of the staging reaches DRAM:
//   v0  16-B stores, evict_last policy (the engine's form)
//   v1  16-B stores, no policy
//   v2  full 32-B sector per store pair (two adjacent lanes fill one sector)
//   v3  v0 after a memset of the staging (sectors already valid in L2)
//   v4  v0 with no L2 flush before it
// Run under ncu with dram__bytes_write.sum to read the per-kernel DRAM bytes.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
#include <algorithm>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t pol_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t pol_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}

template <int V>
__global__ void __launch_bounds__(256) scatter(const double2* __restrict__ x, const uint32_t* __restrict__ pos,
                                               const uint32_t* __restrict__ dst, double2* S, int N) {
  const uint64_t pf = pol_first(), pl = pol_last();
  const int T = gridDim.x * blockDim.x;
  for (int q0 = blockIdx.x * blockDim.x + threadIdx.x; q0 < N; q0 += 8 * T) {
    double2 v[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      const int q = q0 + c * T;
      if (q < N)
        asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.L2::64B.v2.f64 {%0, %1}, [%2], %3;"
                     : "=d"(v[c].x), "=d"(v[c].y) : "l"(x + pos[q]), "l"(pf));
    }
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      const int q = q0 + c * T;
      if (q < N) {
        uint32_t d;
        if (V == 2) d = 2 * dst[q >> 1] + (q & 1);  // lanes 2m, 2m+1 fill one 32-B sector
        else d = dst[q];
        if (V == 1)
          asm volatile("st.global.v2.f64 [%0], {%1, %2};" ::"l"(S + d), "d"(v[c].x), "d"(v[c].y));
        else
          asm volatile("st.global.L2::cache_hint.v2.f64 [%0], {%1, %2}, %3;" ::"l"(S + d), "d"(v[c].x),
                       "d"(v[c].y), "l"(pl));
      }
    }
  }
}

__global__ void readS(const double4* __restrict__ S, size_t n4, double* out) {
  double a = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x) {
    const double4 v = S[i];
    a += v.x + v.y + v.z + v.w;
  }
  if (a == 1.2345) out[0] = a;
}

__global__ void flush_read(const int4* __restrict__ p, size_t n, int* out) {
  int a = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    a ^= p[i].x ^ p[i].w;
  if (a == 12345) out[0] = a;
}

int main() {
  const uint32_t n = 1u << 24;
  const int N = 2800000 & ~1;
  std::mt19937_64 rng(1);
  std::vector<uint32_t> pos(N), dst(N);
  for (auto& p : pos) p = (uint32_t)(rng() % n);
  std::sort(pos.begin(), pos.end());
  for (int i = 0; i < N; ++i) dst[i] = i;
  std::shuffle(dst.begin(), dst.end(), rng);
  std::vector<uint32_t> dst2(N / 2);  // permutation of the N/2 sectors for v2
  for (int i = 0; i < N / 2; ++i) dst2[i] = i;
  std::shuffle(dst2.begin(), dst2.end(), rng);
  double2 *x, *S;
  uint32_t *dpos, *ddst, *ddst2;
  uint8_t* fw;
  int* fo;
  double* o;
  const size_t fb = 256ull << 20;
  cudaMalloc(&x, (size_t)n * 16);
  cudaMalloc(&S, (size_t)N * 16);
  cudaMalloc(&dpos, N * 4);
  cudaMalloc(&ddst, N * 4);
  cudaMalloc(&ddst2, N * 2);
  cudaMalloc(&fw, fb);
  cudaMalloc(&fo, 64);
  cudaMalloc(&o, 64);
  void* fr;
  cudaMalloc(&fr, fb);
  cudaMemset(x, 1, (size_t)n * 16);
  cudaMemset(fr, 1, fb);
  cudaMemcpy(dpos, pos.data(), N * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(ddst, dst.data(), N * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(ddst2, dst2.data(), N * 2, cudaMemcpyHostToDevice);
  const size_t sbytes = (size_t)N * 16;
  cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, sbytes);
  size_t got = 0;
  cudaDeviceGetLimit(&got, cudaLimitPersistingL2CacheSize);
  printf("staging %.1f MB, set-aside %.1f MB\n", sbytes / 1e6, got / 1e6);
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int grid = sms * 4;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  auto flush = [&]() {
    cudaMemsetAsync(fw, 0, fb);
    flush_read<<<sms * 8, 256>>>((const int4*)fr, fb / 16, fo);
  };
  const char* names[] = {"v0 16B evict_last", "v1 16B no hint", "v2 32B sector pairs", "v3 memset first",
                         "v4 no flush"};
  for (int v = 0; v < 5; ++v) {
    float tot = 0, tr = 0;
    const int reps = 6;
    for (int r = 0; r < reps + 2; ++r) {
      if (v != 4) flush();
      if (v == 3) cudaMemsetAsync(S, 0, sbytes);
      cudaEventRecord(a);
      switch (v) {
        case 0: case 3: case 4: scatter<0><<<grid, 256>>>(x, dpos, ddst, S, N); break;
        case 1: scatter<1><<<grid, 256>>>(x, dpos, ddst, S, N); break;
        case 2: scatter<2><<<grid, 256>>>(x, dpos, ddst2, S, N); break;
      }
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      cudaEventRecord(a);
      readS<<<sms * 4, 256>>>((const double4*)S, sbytes / 32, o);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms2;
      cudaEventElapsedTime(&ms2, a, b);
      if (r >= 2) tot += ms, tr += ms2;
    }
    printf("%-22s scatter %.1f us  readS %.1f us\n", names[v], 1e3 * tot / reps, 1e3 * tr / reps);
  }
  cudaError_t e = cudaDeviceSynchronize();
  printf("status %s\n", cudaGetErrorString(e));
  return 0;
}
