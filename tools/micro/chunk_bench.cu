// chunk_bench.cu -- cycles per chunk of the production WaveCompute::chunk<MODE> for one warp with
// fake (always-ready) links.  Development tool.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I../../paper_conf_ipps_kumark15_b200/csrc -o chunk_bench chunk_bench.cu
#include <cstdio>
#include "wavefront.cuh"

using namespace lddp;

template <class F, int R, int SIG, int E, int MODE>
__global__ void bench(FillParams p, int chunks, long long* out) {
  using WC = WaveCompute<F, R, SIG, E, 4, F::kGridIn>;
  using T = typename WC::T;
  __shared__ alignas(16) T top[32];
  __shared__ alignas(16) T bot[32];
  __shared__ typename WC::CC bring[kBRing];
  const int lane = threadIdx.x & 31;
  top[lane] = T(0);
  for (int i = lane; i < kBRing; i += 32) bring[i] = typename WC::CC(F::col_ctx(p, i % 1000));
  __syncwarp();
  WC cs;
  cs.bring = bring;
  cs.carry_tau = INT_MIN;
  for (int r = 0; r < R; ++r) {
    cs.irow[r] = lane * R + r + (MODE == 1 ? -1 : 0);
    cs.rvalid[r] = cs.irow[r] >= 0;
    cs.vtop[r] = cs.irow[r] == -1;
    cs.rc[r] = F::row_ctx(p, cs.rvalid[r] ? cs.irow[r] : 0);
    cs.leftv[r] = T(0);
    cs.rightv[r] = T(0);
    cs.rlast[r] = T(0);
    for (int d = 0; d < WC::HV; ++d) cs.hist[r][d] = T(0);
    for (int d = 0; d < WC::HC; ++d) cs.hcc[r][d] = typename WC::CC(0);
  }
  for (int d = 0; d < WC::FV; ++d) cs.fifo[d] = T(0);
  // steady chunks start at a column where every lane is inside the table
  const int tau0 = (MODE == 2) ? -40 : 32 * WC::D + 64;
  long long t0 = clock64();
  for (int k = 0; k < chunks; ++k) cs.template chunk<MODE>(p, lane, tau0 + (MODE == 2 ? 0 : k * 32), top, bot, true);
  long long t1 = clock64();
  T acc = T(0);
  for (int r = 0; r < R; ++r) acc += cs.hist[r][0];
  if (acc == T(12345)) out[1] = 1;
  if (lane == 0) out[0] = (t1 - t0) / chunks;
}

template <class F, int R, int SIG, int E, int MODE>
void run(const char* name, FillParams p, long long* d) {
  bench<F, R, SIG, E, MODE><<<1, 32>>>(p, 64, d);
  cudaError_t e = cudaDeviceSynchronize();
  long long h = 0;
  cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  printf("%-6s R=%d SIG=%d E=%d MODE=%d: %lld cycles/chunk = %.1f cycles/step %s\n", name, R, SIG, E, MODE, h,
         h / 32.0, e == cudaSuccess ? "" : cudaGetErrorString(e));
}

int main() {
  const int n = 1 << 20;
  uint8_t* b;
  float* y;
  long long* d;
  cudaMalloc(&b, n);
  cudaMalloc(&y, n * 4);
  cudaMalloc(&d, 64);
  cudaMemset(b, 65, n);
  cudaMemset(y, 0, n * 4);
  FillParams p;
  memset(&p, 0, sizeof p);
  p.a = b;
  p.b = b;
  p.rows = 1 << 20;
  p.cols = n - 4096;
  p.cols_total = p.cols;
  run<CellLCS, 4, 0, 2, 0>("LCS", p, d);
  run<CellLCS, 4, 0, 2, 1>("LCS", p, d);
  run<CellLCS, 4, 0, 2, 2>("LCS", p, d);
  run<CellLCS, 4, 1, 1, 0>("LCS", p, d);
  run<CellLCS, 4, 1, 1, 2>("LCS", p, d);
  run<CellLCS, 8, 1, 1, 0>("LCS", p, d);
  run<CellLCS, 2, 1, 1, 0>("LCS", p, d);
  uint8_t* img;
  cudaMalloc(&img, (size_t)4096 * 16384);
  cudaMemset(img, 100, (size_t)4096 * 16384);
  p.grid = img;
  p.grid_pitch = 16384;
  p.cols = 16000;
  uint8_t* outimg;
  cudaMalloc(&outimg, (size_t)4096 * 16384);
  p.table = outimg;
  p.table_pitch = 16384;
  run<CellFS, 1, 2, 2, 0>("FS", p, d);
  run<CellFS, 1, 2, 2, 2>("FS", p, d);
  p.grid_pitch = 0;
  run<CellFS, 1, 2, 2, 0>("FS-in0", p, d);
  p.table_pitch = 0;
  run<CellFS, 1, 2, 2, 0>("FS-io0", p, d);
  p.grid_pitch = 16384;
  run<CellFS, 1, 2, 2, 0>("FS-out0", p, d);
  p.table_pitch = 16384;
  p.cols = n - 4096;
  p.a = y;
  p.b = y;
  run<CellDTW, 4, 0, 2, 0>("DTW", p, d);
  run<CellDTW, 4, 0, 2, 2>("DTW", p, d);
  run<CellDTW, 4, 1, 1, 0>("DTW", p, d);
  return 0;
}
