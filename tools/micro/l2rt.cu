// l2rt.cu -- L2 round trip of the load flavours the edge / boundary exchanges use (one warp,
// dependent chain over an L2-resident buffer, clock64), and the store -> load visibility time
// between two warps on different SMs.  Development / measurement tool.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o l2rt l2rt.cu && ./l2rt
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ void ld_rlx(const uint64_t* p, uint64_t& a, uint64_t& b) {
  asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}
__device__ __forceinline__ void ld_rlx_nm(const uint64_t* p, uint64_t& a, uint64_t& b) {
  asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p));
}
__device__ __forceinline__ void ld_cg(const uint64_t* p, uint64_t& a, uint64_t& b) {
  asm volatile("ld.global.cg.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p));
}

// buf: chain next index in element 0 of each 64-byte line (stride 4 KiB apart -> distinct slices)
__global__ void chase(const uint64_t* buf, int n, long long* out) {
  uint64_t i = 0, b = 0;
  long long t0, t1;
  for (int k = 0; k < 64; ++k) { uint64_t a; ld_cg(buf + i, a, b); i = a + (b & 0); }   // warm
  i = 0;
  t0 = clock64();
  for (int k = 0; k < n; ++k) { uint64_t a; ld_rlx(buf + i, a, b); i = a + (b & 0); }
  t1 = clock64();
  out[0] = (t1 - t0) / n;
  i = 0;
  t0 = clock64();
  for (int k = 0; k < n; ++k) { uint64_t a; ld_rlx_nm(buf + i, a, b); i = a + (b & 0); }
  t1 = clock64();
  out[1] = (t1 - t0) / n;
  i = 0;
  t0 = clock64();
  for (int k = 0; k < n; ++k) { uint64_t a; ld_cg(buf + i, a, b); i = a + (b & 0); }
  t1 = clock64();
  out[2] = (t1 - t0) / n;
  out[7] = (long long)i;
}

// ping-pong between CTA 0 and CTA 1 (different SMs): each waits for the other's counter value,
// then stores the next one: one round = two store -> load visibilities.  MODE selects the store /
// load flavour: 0 st.relaxed.gpu / ld.relaxed.gpu, 1 st.volatile / ld.volatile, 2 st.global.cg /
// ld.global.cg (weak, L2-coherent in practice), 3 atom.exch / atom.or 0 (L2 atomics),
// 4 st.relaxed.gpu / two staggered polling warps, 5 red.release.gpu / ld.acquire.gpu
template <int MODE>
__device__ __forceinline__ void pp_st(uint64_t* p, uint64_t v) {
  if (MODE == 0 || MODE == 4) asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
  if (MODE == 1) asm volatile("st.volatile.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
  if (MODE == 2) asm volatile("st.global.cg.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
  if (MODE == 3) { uint64_t o; asm volatile("atom.relaxed.gpu.global.exch.b64 %0, [%1], %2;" : "=l"(o) : "l"(p), "l"(v) : "memory"); }
  if (MODE == 5) asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
template <int MODE>
__device__ __forceinline__ uint64_t pp_ld(const uint64_t* p) {
  uint64_t v;
  if (MODE == 0 || MODE == 4) asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  if (MODE == 1) asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  if (MODE == 2) asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  if (MODE == 3) asm volatile("atom.relaxed.gpu.global.or.b64 %0, [%1], 0;" : "=l"(v) : "l"(p) : "memory");
  if (MODE == 5) asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
template <int MODE>
__global__ void pingpong(uint64_t* flags, int n, long long* out) {
  const int me = blockIdx.x;
  uint64_t* mine = flags + me * 64;
  uint64_t* other = flags + (1 - me) * 64;
  const int w = threadIdx.x >> 5;
  if ((threadIdx.x & 31) != 0) return;
  if (MODE != 4 && w != 0) return;
  __shared__ volatile int seen;
  if (threadIdx.x == 0) seen = 0;
  __syncthreads();
  long long t0 = clock64();
  for (int k = 0; k < n; ++k) {
    const uint64_t want = (uint64_t)(me == 0 ? 2 * k + 2 : 2 * k + 1);
    if (me == 0 && w == 0) pp_st<MODE>(mine, (uint64_t)(2 * k + 1));
    if (MODE == 4) {
      // two warps poll the same word, the second one offset by ~half a round trip
      if (w == 1) { long long t = clock64(); while (clock64() - t < 150) { } }
      while (seen < k + 1) {
        if (pp_ld<MODE>(other) == want) { seen = k + 1; break; }
      }
    } else {
      while (pp_ld<MODE>(other) != want) { }
    }
    if (me == 1 && w == 0) pp_st<MODE>(mine, (uint64_t)(2 * k + 2));
  }
  long long t1 = clock64();
  if (me == 0 && w == 0) out[MODE] = (t1 - t0) / n;
}

int main() {
  const int N = 1 << 20;
  uint64_t* buf;
  cudaMalloc(&buf, N * 8);
  uint64_t* h = new uint64_t[N]();
  // 256 lines, stride 512 elements (4 KiB), pseudo-random order
  const int L = 256;
  int perm[L];
  for (int k = 0; k < L; ++k) perm[k] = (k * 97) % L;
  for (int k = 0; k < L; ++k) h[(size_t)perm[k] * 512] = (uint64_t)perm[(k + 1) % L] * 512;
  cudaMemcpy(buf, h, N * 8, cudaMemcpyHostToDevice);
  long long* out;
  cudaMalloc(&out, 64);
  cudaMemset(out, 0, 64);
  chase<<<1, 32>>>(buf, 4096, out);
  chase<<<1, 32>>>(buf, 4096, out);
  uint64_t* flags;
  cudaMalloc(&flags, 4096 * 8);
  long long* pout;
  cudaMalloc(&pout, 64);
  cudaMemset(pout, 0, 64);
#define PP(M) cudaMemset(flags, 0, 4096 * 8); pingpong<M><<<2, 64>>>(flags, 2000, pout); cudaDeviceSynchronize();
  PP(0) PP(1) PP(2) PP(3) PP(4) PP(5)
  long long q[8];
  cudaMemcpy(q, pout, 64, cudaMemcpyDeviceToHost);
  printf("{\"pingpong_round\": {\"relaxed_gpu\": %lld, \"volatile\": %lld, \"cg\": %lld, \"atomics\": %lld, "
         "\"relaxed_2pollers\": %lld, \"release_acquire\": %lld}, \"unit\": \"SM cycles per round (2 one-way visibilities)\"}\n",
         q[0], q[1], q[2], q[3], q[4], q[5]);
  long long r[8];
  cudaMemcpy(r, out, 64, cudaMemcpyDeviceToHost);
  printf("{\"ld_relaxed_gpu_v2\": %lld, \"ld_relaxed_gpu_v2_noclobber\": %lld, \"ld_cg_v2\": %lld, "
         "\"unit\": \"SM cycles per dependent load\", \"how\": \"tools/micro/l2rt.cu\"}\n", r[0], r[1], r[2]);
  return 0;
}
