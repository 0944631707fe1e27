// Microbenchmark (experiment, not product): dependent random 8-byte shared-memory loads, the
// per-visit cost of a tree-stationary walk where the 32 lanes of a warp are at unrelated nodes of
// the resident trees.  Each lane follows K independent chains through a random permutation of
// N uint2 words (y = next index); reads/s over all SMs.  Also a variant with a second, dependent
// 4-byte load from a lane-private (conflict-free) column per step (the row attribute read).
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
#include <algorithm>
#include <cuda_runtime.h>

template <int K, bool ATTR>
__global__ void __launch_bounds__(1024, 1) walk(const uint2* __restrict__ g, int N, int steps, unsigned long long* sink) {
  extern __shared__ uint2 s[];
  for (int i = threadIdx.x; i < N; i += blockDim.x) s[i] = g[i];
  float* attr = reinterpret_cast<float*>(s + N);   // [64][1024 lanes]: lane-private columns
  for (int i = threadIdx.x; i < 64 * 32; i += blockDim.x) attr[i] = (float)i;
  __syncthreads();
  uint32_t p[K];
  for (int k = 0; k < K; k++) p[k] = (threadIdx.x * 7919u + k * 104729u + blockIdx.x * 31u) % (uint32_t)N;
  float acc = 0.f;
  const int lane = threadIdx.x & 31;
  for (int it = 0; it < steps; it++) {
#pragma unroll
    for (int k = 0; k < K; k++) {
      uint2 w = s[p[k]];
      if (ATTR) {
        float a = attr[(w.x & 63) * 32 + lane];
        p[k] = a < 1e9f ? w.y : w.x;
      } else {
        p[k] = w.y;
        acc += __uint_as_float(w.x);
      }
    }
  }
  uint32_t h = 0;
  for (int k = 0; k < K; k++) h ^= p[k];
  if (h == 0x12345678u && acc == 1.0f) sink[blockIdx.x] = h;
}

template <int K, bool ATTR>
double run(int N, int sms) {
  std::vector<uint32_t> perm(N);
  for (int i = 0; i < N; i++) perm[i] = i;
  std::mt19937 rng(1);
  std::shuffle(perm.begin(), perm.end(), rng);
  std::vector<uint2> h(N);
  for (int i = 0; i < N; i++) h[perm[i]] = make_uint2(perm[(i + 1) % N] , perm[(i + 1) % N]);
  uint2* d; unsigned long long* sink;
  cudaMalloc(&d, N * 8); cudaMalloc(&sink, 8 * sms);
  cudaMemcpy(d, h.data(), N * 8, cudaMemcpyHostToDevice);
  int smem = N * 8 + 64 * 32 * 4;
  cudaFuncSetAttribute(walk<K, ATTR>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int steps = 4096 / K;
  walk<K, ATTR><<<sms, 1024, smem>>>(d, N, steps / 8, sink);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  walk<K, ATTR><<<sms, 1024, smem>>>(d, N, steps, sink);
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) printf("err %s\n", cudaGetErrorString(e));
  cudaFree(d); cudaFree(sink);
  return (double)sms * 1024.0 * steps * K / (ms / 1e3);
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (int N : {2048, 16384, 24000}) {
    printf("N=%d words: K=1 %.3g  K=2 %.3g  K=4 %.3g reads/s | +attr K=2 %.3g K=4 %.3g\n", N,
           run<1, false>(N, sms), run<2, false>(N, sms), run<4, false>(N, sms), run<2, true>(N, sms), run<4, true>(N, sms));
  }
  return 0;
}
