// Fixed-cost calibration: empty kernels vs dynamic smem, syncthreads cost, L2 latency.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void empty_k(int* p) { extern __shared__ int s[]; if (threadIdx.x == 9999) p[0] = s[0]; }
__global__ void syncs_k(int* p, int n) {
  __shared__ int s[1024];
  int v = threadIdx.x;
  for (int i = 0; i < n; ++i) { s[threadIdx.x] = v; __syncthreads(); v += s[(threadIdx.x + 1) & 1023]; __syncthreads(); }
  if (v == -1) p[0] = v;
}
__global__ void chase_k(const int* __restrict__ nxt, int* out, int n) {
  int j = 0;
  for (int i = 0; i < n; ++i) j = nxt[j];
  out[0] = j;
}
template <class F> float t_graph(F launch, int reps) {
  cudaStream_t s; cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaGraph_t g; cudaGraphExec_t e;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
  for (int i = 0; i < reps; ++i) launch(s);
  cudaStreamEndCapture(s, &g); cudaGraphInstantiate(&e, g, 0);
  cudaGraphLaunch(e, s); cudaStreamSynchronize(s);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a, s); cudaGraphLaunch(e, s); cudaEventRecord(b, s); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b); return ms * 1e3f / reps;
}
int main() {
  int* p; cudaMalloc(&p, 1 << 26);
  for (int smem : {0, 16384, 65536, 131072, 200000}) {
    cudaFuncSetAttribute(empty_k, cudaFuncAttributeMaxDynamicSharedMemorySize, 220000);
    for (int thr : {128, 1024}) for (int grid : {1, 8, 148, 592}) {
      float us = t_graph([&](cudaStream_t s) { empty_k<<<grid, thr, smem, s>>>(p); }, 200);
      printf("empty smem=%6d thr=%4d grid=%4d : %.2f us/launch\n", smem, thr, grid, us);
    }
  }
  // alternating smem sizes (carveout reconfiguration)
  float us = t_graph([&](cudaStream_t s) { empty_k<<<148, 1024, 0, s>>>(p); empty_k<<<148, 1024, 200000, s>>>(p); }, 100);
  printf("alternating 0/200000 smem: %.2f us per pair\n", us);
  for (int n : {1, 10, 100}) {
    float t = t_graph([&](cudaStream_t s) { syncs_k<<<1, 1024, 0, s>>>(p, n); }, 50);
    printf("syncs 1024 thr n=%d (2 syncs each): %.2f us\n", n, t);
  }
  // pointer chase in L2 (4 MB buffer, random-ish stride)
  int N = 1 << 20; int* h = new int[N];
  for (int i = 0; i < N; ++i) h[i] = (int)(((long long)i * 7919 + 104729) % N);
  int* d; cudaMalloc(&d, N * 4); cudaMemcpy(d, h, N * 4, cudaMemcpyHostToDevice);
  for (int n : {100, 1000}) {
    float t = t_graph([&](cudaStream_t s) { chase_k<<<1, 1, 0, s>>>(d, p, n); }, 10);
    printf("chase n=%d: %.2f us -> %.1f ns/load\n", n, t, t * 1e3 / n);
  }
  return 0;
}
