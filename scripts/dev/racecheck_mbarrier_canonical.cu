// Does compute-sanitizer racecheck model mbarrier arrive(release) / try_wait(acquire) as
// synchronization?  Two canonical hand-offs, each correct under the PTX memory model:
//   A: warp 0 writes shared memory, arrives (release) on an mbarrier; warp 1 waits (acquire), reads.
//   B: the same with a __syncthreads() instead of the mbarrier (control).
//   C: as A, but after __syncwarp() only lane 0 arrives (count 1) for the whole warp — equally
//      ordered by the PTX memory model (bar.warp.sync orders the lanes' writes before lane 0's
//      release).
//   D: two TMA bulk copies into the same shared buffer issued by DIFFERENT threads, the second
//      only after its thread has waited (acquire) on the mbarrier the first copy completed —
//      ordered by the memory model (complete_tx -> try_wait.acquire -> fence.proxy.async).
// nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/rc racecheck_mbarrier_canonical.cu
// compute-sanitizer --tool racecheck /tmp/rc A   |   ... /tmp/rc B
#include <cstdio>
#include <cstdint>
#include <cstring>

__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void k(int mode, int* out, const int* src) {
  __shared__ uint64_t bar;
  __shared__ uint64_t bar2;
  __shared__ __align__(128) int buf[32];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (mode == 3) {
    if (threadIdx.x == 0) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&bar)) : "memory");
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&bar2)) : "memory");
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x == 0) {   // warp 0: first copy
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], 128;" ::"r"(sa(&bar)) : "memory");
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 128, [%2];" ::"r"(sa(buf)), "l"(src), "r"(sa(&bar)) : "memory");
    }
    if (threadIdx.x == 32) {  // warp 1: waits for the first copy, then overwrites the buffer
      asm volatile("{\n\t.reg .pred p;\nW3:\n\tmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%0], 0;\n\t@!p bra W3;\n}" ::"r"(sa(&bar)) : "memory");
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], 128;" ::"r"(sa(&bar2)) : "memory");
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 128, [%2];" ::"r"(sa(buf)), "l"(src + 32), "r"(sa(&bar2)) : "memory");
      asm volatile("{\n\t.reg .pred p;\nW4:\n\tmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%0], 0;\n\t@!p bra W4;\n}" ::"r"(sa(&bar2)) : "memory");
      out[0] = buf[31];
    }
    return;
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(&bar)), "r"(mode == 2 ? 1 : 32) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (mode == 0 || mode == 2) {
    if (warp == 0) {
      buf[lane] = lane * 3;
      if (mode == 2) __syncwarp();
      if (mode == 0 || lane == 0)
        asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(sa(&bar)) : "memory");
    } else {
      asm volatile("{\n\t.reg .pred p;\nW:\n\tmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%0], 0;\n\t@!p bra W;\n}" ::"r"(sa(&bar)) : "memory");
      out[lane] = buf[31 - lane];
    }
  } else {
    if (warp == 0) buf[lane] = lane * 3;
    __syncthreads();
    if (warp == 1) out[lane] = buf[31 - lane];
  }
}

int main(int argc, char** argv) {
  const int mode = (argc > 1 && !strcmp(argv[1], "B")) ? 1 : (argc > 1 && !strcmp(argv[1], "C")) ? 2
                 : (argc > 1 && !strcmp(argv[1], "D")) ? 3 : 0;
  int* d;
  int* src;
  cudaMalloc(&d, 128);
  cudaMalloc(&src, 256);
  int hs[64];
  for (int i = 0; i < 64; i++) hs[i] = i < 32 ? 0 : 93 * (i == 63);
  cudaMemcpy(src, hs, 256, cudaMemcpyHostToDevice);
  k<<<1, 64>>>(mode, d, src);
  int h[32];
  cudaMemcpy(h, d, 128, cudaMemcpyDeviceToHost);
  printf("mode %s: out[0] = %d (expect 93)\n", mode == 1 ? "B (syncthreads)" : mode == 2 ? "C (lane-0 arrive)" : mode == 3 ? "D (TMA after TMA, two threads)" : "A (mbarrier)", h[0]);
  return h[0] == 93 ? 0 : 1;
}
