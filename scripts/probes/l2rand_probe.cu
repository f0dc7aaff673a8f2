// Random 16-B reads from an L2-resident buffer: how many per second?
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__global__ void __launch_bounds__(256) rnd(const double2* __restrict__ buf, uint32_t mask, double2* out, int per) {
  uint32_t h = (blockIdx.x * blockDim.x + threadIdx.x) * 2654435761u + 12345u;
  double ax = 0, ay = 0;
  for (int it = 0; it < per; it += 8) {
    double2 v[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) { h = h * 1664525u + 1013904223u; v[c] = __ldcg(buf + ((h >> 4) & mask)); }
#pragma unroll
    for (int c = 0; c < 8; ++c) { ax += v[c].x; ay += v[c].y; }
  }
  if (ax == 12345.0) out[0] = make_double2(ax, ay);
}
int main() {
  double2 *buf, *out; cudaMalloc(&buf, 1ull << 30); cudaMalloc(&out, 64); cudaMemset(buf, 0, 1ull << 30);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int mb : {8, 16, 32, 48, 64, 96, 128, 512}) {
    uint32_t elems = (uint32_t)((size_t)mb << 20) / 16, mask = elems - 1;
    if (mb == 48) mask = (32u << 20) / 16 - 1;  // keep power of two for mask
    if (mb == 96) mask = (64u << 20) / 16 - 1;
    int grid = 148 * 8, per = 64;
    long long reqs = (long long)grid * 256 * per;
    for (int rep = 0; rep < 3; ++rep) {
      rnd<<<grid, 256>>>(buf, mask, out, per);  // warm
      cudaEventRecord(a); rnd<<<grid, 256>>>(buf, mask, out, per); cudaEventRecord(b); cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b);
      if (rep == 2) printf("buffer %4d MB: %.1f G random 16-B reads/s (%.2f ms for %lld)\n", (int)(((size_t)mask + 1) * 16 >> 20), reqs / (ms * 1e-3) / 1e9, ms, reqs);
    }
  }
  return 0;
}
