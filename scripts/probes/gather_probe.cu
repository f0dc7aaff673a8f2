// Random 16-B gather microbenchmark: which load flavour moves the fewest DRAM bytes?
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
template <int MODE>
__device__ __forceinline__ double2 ld(const double2* p) {
  double2 v;
  if (MODE == 0) asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  if (MODE == 1) asm volatile("ld.global.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  if (MODE == 2) asm volatile("ld.global.cg.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  if (MODE == 3) asm volatile("ld.global.cv.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  if (MODE == 4) asm volatile("ld.global.nc.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  if (MODE == 5) asm volatile("ld.global.L1::no_allocate.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  if (MODE == 6) asm volatile("ld.global.lu.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  if (MODE == 7) asm volatile("ld.global.nc.L1::no_allocate.L2::64B.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  return v;
}
template <int MODE>
__global__ void __launch_bounds__(256) gather(const double2* __restrict__ x, double2* out, uint32_t nmask, int B, int R) {
  int j = blockIdx.x * blockDim.x + threadIdx.x;
  uint32_t sigma = 0x9E3779B1u | 1u, tau = blockIdx.y * 7919u;
  sigma += blockIdx.y * 2654435761u * 2u;
  double ar = 0, ai = 0;
  double2 v[13];
#pragma unroll
  for (int c = 0; c < 13; ++c) {
    uint32_t i = j + c * B;
    v[c] = ld<MODE>(x + ((sigma * i + tau) & nmask));
  }
#pragma unroll
  for (int c = 0; c < 13; ++c) { ar += v[c].x; ai += v[c].y; }
  out[blockIdx.y * B + j] = make_double2(ar, ai);
}
template <int MODE>
float run(const double2* x, double2* out, char* flush, uint32_t nmask) {
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  float best = 1e9;
  for (int it = 0; it < 6; ++it) {
    cudaMemset(flush, it, 512u << 20);
    cudaEventRecord(a);
    gather<MODE><<<dim3(64, 16), 256>>>(x, out, nmask, 16384, 13);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float t; cudaEventElapsedTime(&t, a, b); if (it > 0 && t < best) best = t;
  }
  return best;
}
int main() {
  size_t n = 1u << 24;
  double2 *x, *out; char* flush;
  cudaMalloc(&x, n * 16); cudaMalloc(&out, 16 * 16384 * 16); cudaMalloc(&flush, 512u << 20);
  cudaMemset(x, 0, n * 16);
  printf("mode0 nc.L1::no_allocate %.2f us\n", 1e3 * run<0>(x, out, flush, n - 1));
  printf("mode1 plain              %.2f us\n", 1e3 * run<1>(x, out, flush, n - 1));
  printf("mode2 cg                 %.2f us\n", 1e3 * run<2>(x, out, flush, n - 1));
  printf("mode3 cv                 %.2f us\n", 1e3 * run<3>(x, out, flush, n - 1));
  printf("mode4 nc                 %.2f us\n", 1e3 * run<4>(x, out, flush, n - 1));
  printf("mode5 L1::no_allocate    %.2f us\n", 1e3 * run<5>(x, out, flush, n - 1));
  printf("mode6 lu                 %.2f us\n", 1e3 * run<6>(x, out, flush, n - 1));
  printf("mode7 nc L2::64B         %.2f us\n", 1e3 * run<7>(x, out, flush, n - 1));
  return 0;
}
