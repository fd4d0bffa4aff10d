// tma_box.cu -- one 2-D tensor-TMA box load (int32, zero OOB fill) per launch with a given box
// origin and width, to check which box geometries the TMA unit accepts.  Development tool.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o tma_box tma_box.cu && ./tma_box
#include <cstdio>
#include <cstring>
#include <cstdint>
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

__global__ void k(const __grid_constant__ CUtensorMap tm, int x, int y, int bytes, int* out) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ __align__(8) uint64_t bar;
  const uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar);
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(sm);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(bytes) : "memory");
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(d),
        "l"(reinterpret_cast<uint64_t>(&tm)), "r"(x), "r"(y), "r"(b)
        : "memory");
    uint32_t ok = 0;
    while (!ok) {
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(ok) : "r"(b) : "memory");
    }
    out[0] = reinterpret_cast<int*>(sm)[0];
    out[1] = reinterpret_cast<int*>(sm)[1];
  }
}

int main() {
  const int H = 300, W = 300;
  int* g;
  cudaMalloc(&g, H * W * 4);
  int* h = new int[H * W];
  for (int i = 0; i < H * W; ++i) h[i] = i;
  cudaMemcpy(g, h, H * W * 4, cudaMemcpyHostToDevice);
  int* out;
  cudaMalloc(&out, 64);
  void* fp = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fp, cudaEnableDefault, &q);
  auto enc = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fp);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 100000);
  const int cases[][4] = {{64, 32, 0, 0}, {64, 32, -31, 204}, {128, 32, -32, 0}, {64, 32, 250, 10}, {64, 32, 299, 299},
                          {64, 32, 400, 0}, {32, 32, 0, 0}, {64, 16, 0, 0}};
  for (auto& c : cases) {
    CUtensorMap tm;
    memset(&tm, 0, sizeof tm);
    const cuuint64_t dims[2] = {(cuuint64_t)W, (cuuint64_t)H};
    const cuuint64_t strides[1] = {(cuuint64_t)W * 4};
    const cuuint32_t box[2] = {(cuuint32_t)c[0], (cuuint32_t)c[1]};
    const cuuint32_t es[2] = {1, 1};
    CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_INT32, 2, g, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    k<<<1, 32, c[0] * c[1] * 4>>>(tm, c[2], c[3], c[0] * c[1] * 4, out);
    cudaError_t e = cudaDeviceSynchronize();
    int o[2] = {-1, -1};
    if (e == cudaSuccess) cudaMemcpy(o, out, 8, cudaMemcpyDeviceToHost);
    printf("box %dx%d at (%d,%d): encode %d, run %s, first %d %d\n", c[0], c[1], c[2], c[3], (int)r,
           cudaGetErrorString(e), o[0], o[1]);
    if (e != cudaSuccess) return 1;
  }
  return 0;
}
