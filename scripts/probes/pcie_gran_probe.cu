// Zero-copy read rate from pinned host memory by request granularity: is the
// in-place PCIe gather of cusfft_execute_host (C3: 1.66M distinct 32-B sectors
// of a 256 MB x, 2.27 ms) bound by bytes or by the number of read requests?
// Reads M distinct G-byte chunks (G = 32 / 64 / 128, aligned, random order,
// positions sorted like the staged gather's address-ordered schedule or
// shuffled) of a 256 MB pinned buffer; one G-byte chunk per group of G/16
// threads (16-B loads, one request per chunk).  Prints ms, chunks/s, GB/s.
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/pg pcie_gran_probe.cu
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <random>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e_)); exit(1); } } while (0)

template <int G>
__global__ void k_read(const uint4* __restrict__ x, const uint32_t* __restrict__ chunk, int m, uint4* __restrict__ sink) {
  constexpr int TPC = G / 16;  // threads per chunk
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  uint4 acc = make_uint4(0, 0, 0, 0);
  for (int64_t i = t; i < (int64_t)m * TPC; i += stride) {
    const uint32_t c = __ldg(chunk + i / TPC);
    uint4 v;
    asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                 : "l"(x + (int64_t)c * TPC + (i % TPC)));
    acc.x ^= v.x; acc.y ^= v.y; acc.z ^= v.z; acc.w ^= v.w;
  }
  if ((acc.x ^ acc.y ^ acc.z ^ acc.w) == 0x9e3779b9u) sink[0] = acc;
}

template <int G>
float run(const uint4* xh, const uint32_t* d_chunk, int m, uint4* sink, int blocks, int threads) {
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a));
  CK(cudaEventCreate(&b));
  k_read<G><<<blocks, threads>>>(xh, d_chunk, m, sink);
  CK(cudaDeviceSynchronize());
  float best = 1e30f;
  for (int r = 0; r < 5; ++r) {
    CK(cudaEventRecord(a));
    k_read<G><<<blocks, threads>>>(xh, d_chunk, m, sink);
    CK(cudaEventRecord(b));
    CK(cudaEventSynchronize(b));
    float ms;
    CK(cudaEventElapsedTime(&ms, a, b));
    best = std::min(best, ms);
  }
  return best;
}

int main() {
  const size_t nbytes = size_t(256) << 20;  // C3's x: 2^24 complex fp64
  void* xh_raw = nullptr;
  CK(cudaHostAlloc(&xh_raw, nbytes, cudaHostAllocMapped));
  memset(xh_raw, 1, nbytes);
  uint4* xh = nullptr;
  CK(cudaHostGetDevicePointer((void**)&xh, xh_raw, 0));
  uint4* sink;
  CK(cudaMalloc(&sink, 64));
  uint32_t* d_chunk;
  const int mmax = 1656683;  // C3's distinct 32-B sectors
  CK(cudaMalloc(&d_chunk, sizeof(uint32_t) * mmax));
  std::mt19937_64 rng(7);
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  printf("G_bytes order chunks ms Mchunks_per_s GB_per_s (payload) threads\n");
  for (int G : {32, 64, 128}) {
    const uint32_t nch = (uint32_t)(nbytes / G);
    for (int m : {mmax, mmax * 3 / 4, mmax / 2}) {
      // m distinct chunks: a random subset of all chunks
      std::vector<uint32_t> all(nch);
      for (uint32_t i = 0; i < nch; ++i) all[i] = i;
      for (int i = 0; i < m; ++i) std::swap(all[i], all[i + rng() % (nch - i)]);
      std::vector<uint32_t> c(all.begin(), all.begin() + m);
      for (int order = 0; order < 2; ++order) {
        if (order == 0) std::sort(c.begin(), c.end());
        else std::shuffle(c.begin(), c.end(), rng);
        CK(cudaMemcpy(d_chunk, c.data(), sizeof(uint32_t) * m, cudaMemcpyHostToDevice));
        for (int tpb : {256}) {
          const int blocks = sms * 8;
          float ms = G == 32 ? run<32>(xh, d_chunk, m, sink, blocks, tpb)
                   : G == 64 ? run<64>(xh, d_chunk, m, sink, blocks, tpb)
                             : run<128>(xh, d_chunk, m, sink, blocks, tpb);
          printf("%d %s %d %.3f %.1f %.2f %d\n", G, order ? "shuffled" : "sorted", m, ms, m / ms / 1e3,
                 (double)m * G / ms / 1e6, blocks * tpb);
        }
      }
    }
  }
  return 0;
}
