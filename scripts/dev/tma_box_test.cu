// Standalone check of a 2-D fp32 tensor-map copy (box W x 32 rows) into dynamic shared memory
// (debugging the TMA-staged wide-code pre-pass).  nvcc -gencode arch=compute_100a,code=sm_100a
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
struct alignas(64) Args { CUtensorMap tmap; int x0, y0, W, off; float* out; };
__global__ void k(const __grid_constant__ Args a) {
  extern __shared__ __align__(1024) float s[];
  uint64_t* bar = reinterpret_cast<uint64_t*>(s + a.off / 4 + a.W * 32);
  uint32_t sb = (uint32_t)__cvta_generic_to_shared(bar);
  uint32_t sd = (uint32_t)__cvta_generic_to_shared(s + a.off / 4);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sb));
    asm volatile("fence.mbarrier_init.release.cluster;");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sb), "r"(a.W * 32 * 4));
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                 ::"r"(sd), "l"(reinterpret_cast<uint64_t>(&a.tmap)), "r"(a.x0), "r"(a.y0), "r"(sb) : "memory");
    asm volatile("{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W;\n}" ::"r"(sb));
    for (int i = 0; i < a.W * 32; i++) a.out[i] = s[a.off / 4 + i];
  }
}
typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                        const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
int main() {
  void* p; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  Enc enc = (Enc)p;
  int d = 600, n = 1000;
  std::vector<float> h((size_t)n * d);
  for (size_t i = 0; i < h.size(); i++) h[i] = (float)i;
  float *X, *out; cudaMalloc(&X, h.size() * 4); cudaMemcpy(X, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  cudaMalloc(&out, 256 * 32 * 4);
  for (int W : {256}) for (int x0 : {40, 41, 42, 66, 400, 599}) for (int l2 : {1}) for (int off : {130048}) for (int thr : {1024}) {
    Args a{}; a.x0 = x0; a.y0 = 100; a.W = W; a.out = out; a.off = off;
    cuuint64_t gdim[2] = {(cuuint64_t)d, (cuuint64_t)n}, gstr[1] = {(cuuint64_t)d * 4};
    cuuint32_t box[2] = {(cuuint32_t)W, 32}, es[2] = {1, 1};
    CUresult r = enc(&a.tmap, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, X, gdim, gstr, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_NONE, l2 ? CU_TENSOR_MAP_L2_PROMOTION_L2_256B : CU_TENSOR_MAP_L2_PROMOTION_NONE,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    int smem = off + 2 * W * 32 * 4 + 64;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    k<<<1, thr, smem>>>(a);
    cudaError_t e = cudaDeviceSynchronize();
    float v[2] = {0, 0}; if (e == cudaSuccess) cudaMemcpy(v, out, 8, cudaMemcpyDeviceToHost);
    printf("off=%d thr=%d W=%d x0=%d l2=%d encode=%d kernel=%s first=%g expect=%g\n", off, thr, W, x0, l2, (int)r, cudaGetErrorString(e), v[0], (float)(100 * d + x0));
    if (e != cudaSuccess) { cudaDeviceReset(); cudaMalloc(&X, h.size() * 4); cudaMemcpy(X, h.data(), h.size() * 4, cudaMemcpyHostToDevice); cudaMalloc(&out, 256 * 32 * 4); }
  }
  return 0;
}
