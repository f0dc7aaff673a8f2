// Random-access-rate probe: 16-B random vs 64-B random vs address-sorted gathers.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>
__device__ __forceinline__ double2 ldnc(const double2* p) {
  double2 v;
  asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  return v;
}
// same index function as gather_probe mode 0
__device__ __forceinline__ uint32_t idx_of(uint32_t j, int c, int y, uint32_t nmask) {
  uint32_t sigma = (0x9E3779B1u | 1u) + y * 2654435761u * 2u, tau = y * 7919u;
  return (sigma * (j + c * 16384u) + tau) & nmask;
}
template <int W>  // W complex elements per random access (1 = 16 B, 4 = 64 B)
__global__ void __launch_bounds__(256) rnd(const double2* __restrict__ x, double2* out, uint32_t nmask) {
  int j = blockIdx.x * blockDim.x + threadIdx.x;
  double ar = 0, ai = 0;
  double2 v[13][W];
#pragma unroll
  for (int c = 0; c < 13; ++c) {
    uint32_t p = idx_of(j, c, blockIdx.y, nmask) & ~(uint32_t)(W - 1);
#pragma unroll
    for (int e = 0; e < W; ++e) v[c][e] = ldnc(x + p + e);
  }
#pragma unroll
  for (int c = 0; c < 13; ++c)
#pragma unroll
    for (int e = 0; e < W; ++e) { ar += v[c][e].x; ai += v[c][e].y; }
  out[blockIdx.y * 16384 + j] = make_double2(ar, ai);
}
// sorted: thread t handles sorted positions t + c*T (coalesced index reads)
__global__ void __launch_bounds__(256) srt(const double2* __restrict__ x, const uint32_t* __restrict__ pos, double2* out, int total) {
  int t = blockIdx.x * blockDim.x + threadIdx.x;
  int T = gridDim.x * blockDim.x;
  double ar = 0, ai = 0;
  double2 v[13];
#pragma unroll
  for (int c = 0; c < 13; ++c) {
    int q = t + c * T;
    v[c] = q < total ? ldnc(x + __ldg(pos + q)) : make_double2(0, 0);
  }
#pragma unroll
  for (int c = 0; c < 13; ++c) { ar += v[c].x; ai += v[c].y; }
  out[t] = make_double2(ar, ai);
}
// sorted, warp-contiguous: warp w handles a contiguous run of 32*13 sorted positions
__global__ void __launch_bounds__(256) srt2(const double2* __restrict__ x, const uint32_t* __restrict__ pos, double2* out, int total) {
  int t = blockIdx.x * blockDim.x + threadIdx.x;
  int warp = t >> 5, lane = t & 31;
  double ar = 0, ai = 0;
  double2 v[13];
#pragma unroll
  for (int c = 0; c < 13; ++c) {
    int q = warp * 32 * 13 + c * 32 + lane;
    v[c] = q < total ? ldnc(x + __ldg(pos + q)) : make_double2(0, 0);
  }
#pragma unroll
  for (int c = 0; c < 13; ++c) { ar += v[c].x; ai += v[c].y; }
  out[t] = make_double2(ar, ai);
}
float timeit(void (*f)(void*), void* arg, char* flush) {
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  float best = 1e9;
  for (int it = 0; it < 6; ++it) {
    cudaMemset(flush, it, 512u << 20);
    cudaEventRecord(a); f(arg); cudaEventRecord(b); cudaEventSynchronize(b);
    float t; cudaEventElapsedTime(&t, a, b); if (it > 0 && t < best) best = t;
  }
  return best * 1e3f;
}
struct Args { double2* x; double2* out; uint32_t* pos; int total; uint32_t nmask; };
int main() {
  size_t n = 1u << 24;
  uint32_t nmask = n - 1;
  double2 *x, *out; char* flush; uint32_t* pos;
  cudaMalloc(&x, n * 16); cudaMalloc(&out, 64u << 20); cudaMalloc(&flush, 512u << 20);
  cudaMemset(x, 0, n * 16);
  // host copy of the index set
  std::vector<uint32_t> h;
  for (int y = 0; y < 16; ++y) for (uint32_t j = 0; j < 16384; ++j) for (int c = 0; c < 13; ++c) {
    uint32_t sigma = (0x9E3779B1u | 1u) + y * 2654435761u * 2u, tau = y * 7919u;
    h.push_back((sigma * (j + c * 16384u) + tau) & nmask);
  }
  std::sort(h.begin(), h.end());
  int total = h.size();
  cudaMalloc(&pos, total * 4);
  cudaMemcpy(pos, h.data(), total * 4, cudaMemcpyHostToDevice);
  Args A{x, out, pos, total, nmask};
  printf("random 16B   : %.2f us\n", timeit([](void* p){ Args* a=(Args*)p; rnd<1><<<dim3(64,16),256>>>(a->x,a->out,a->nmask);}, &A, flush));
  printf("random 32B   : %.2f us\n", timeit([](void* p){ Args* a=(Args*)p; rnd<2><<<dim3(64,16),256>>>(a->x,a->out,a->nmask);}, &A, flush));
  printf("random 64B   : %.2f us\n", timeit([](void* p){ Args* a=(Args*)p; rnd<4><<<dim3(64,16),256>>>(a->x,a->out,a->nmask);}, &A, flush));
  printf("sorted strided: %.2f us\n", timeit([](void* p){ Args* a=(Args*)p; int T=(a->total+12)/13; srt<<<(T+255)/256,256>>>(a->x,a->pos,a->out,a->total);}, &A, flush));
  printf("sorted warprun: %.2f us\n", timeit([](void* p){ Args* a=(Args*)p; int T=(a->total+12)/13; srt2<<<(T+255)/256,256>>>(a->x,a->pos,a->out,a->total);}, &A, flush));
  printf("total %d\n", total);
  return 0;
}
