// fsk.cu -- lane-systolic persistent kernel for Floyd-Steinberg dithering in the knight-move
// category (t = 2i + j, Fig. 2 [L117-L122], Table I row "Y Y Y Y" [L140]; the FS algorithm of
// §VI.B [L341] with the dependency constraint [L343-L344]).  The default FS kernel when the image
// width and row pitch are multiples of 16 bytes (wavefront.cuh is the fallback).
//
//  * STRIPS of SH = 32*W*R rows (top-aligned; rows >= H are computed but never stored).  A CTA of
//    W warps claims strips in increasing order; lane k of warp w owns R rows and processes column
//    c = tau - D*k - 2r for its row r at warp step tau, D = 2R + E: the knight-move skew of 2
//    columns per row plus E steps of slack for the rotate SHFL that carries the lane's last
//    row to the lane below.  Rows r >= 1 take UR / U / UL from row r-1's 3-step error history.
//    Default W = 1, R = 1, E = 1 (measured best: every handoff through global boundary rows).
//  * Row 0 of lane k receives e(i-1, .) from lane k-1 through that one SHFL per step into a
//    register FIFO: UR = fifo[E], U = fifo[E+1], UL = fifo[E+2]; L is the row's previous error.
//    Lane 31 injects the warp's top row (the previous warp's bottom row) into the same SHFL, its
//    8 values per group loaded from shared memory one group ahead.
//  * Pixel arithmetic = CellFS::f, the oracle's pull form and operation order
//    ((((in + e_UL/16) + e_U*5/16) + e_UR*3/16) + e_L*7/16, threshold 128, e = v - out), built
//    with --fmad=false: bit-exact.  Absent neighbours are errors of +0 (v + (+0) == v exactly).
//  * Image rows stream through a per-(lane, row) shared ring of 16-byte chunks (cp.async, 6 chunks
//    ahead), read one 8-step group ahead and converted by mantissa insertion (no I2F); output
//    bytes are collected in a per-row 4-chunk ring and stored 16 bytes at a time.
//  * Warp and strip handoffs of the error rows are the adiag protocol (adiag.cuh): tagged
//    (value, tag) pairs in a shared ring (warp w -> w+1) or in global memory (strip s -> s+1),
//    validated per 32-column chunk; no flags, no fences.
#include <cstdint>
#include <climits>
#include "adiag.cuh"

namespace lddp {

#ifndef LDDP_FSK_PG
#define LDDP_FSK_PG 2   // group of a chunk at which the next chunk's strip-boundary pair is loaded
#endif
namespace {
constexpr int kFsIn = 8;     // input chunks (16 B) per lane ring
constexpr int kFsAhead = 6;  // chunks issued ahead of the lane's current chunk
constexpr int kFsOut = 4;    // output chunks per lane ring

// byte -> float without I2F (a quarter-rate XU op on the step's critical path): the byte as the
// low mantissa bits of 2^23, minus 2^23 -- exact for 0..255, so bit-identical to (float)byte.
__device__ __forceinline__ float fs_u8f(uint32_t byte) {
  return __fsub_rn(__uint_as_float(0x4B000000u | byte), 8388608.0f);
}
__device__ __forceinline__ void fs_cp16(uint32_t dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
}  // namespace

template <int W, int E, int R = 1>
__global__ void __launch_bounds__(W * 32, 1) fsk_kernel(const FillParams p) {
  // R rows per lane, skewed 2 columns apart inside the lane (independent pixels in a step);
  // lane lag D = 2R + E; chunk step origin OFS = 2 + E (lane 31 injects top column tau + OFS)
  constexpr int D = 2 * R + E;
  constexpr int OFS = 2 + E;
  constexpr int SH = W * 32 * R;
  using F = CellFS;
  __shared__ __align__(16) uint64_t ring[W][kAdRing][32];     // top stream of warp w >= 1
  __shared__ int cons[W];
  __shared__ __align__(16) float stg[W][32];                   // bottom staging row
  __shared__ __align__(16) float tstg[W][32];                  // top row of the current chunk
  __shared__ __align__(16) uint8_t inr[W][32][R][kFsIn][16];   // per-(lane, row) input chunks
  __shared__ __align__(16) uint8_t outr[W][32][R][kFsOut][16]; // per-(lane, row) output chunks
  __shared__ int strip_sh;

  Control* ctl = static_cast<Control*>(p.ctl);
  const int lane = threadIdx.x & 31;
  const int wid = threadIdx.x >> 5;
  const int Wimg = p.cols;
  const int64_t H = p.rows;
  const int NQ = (Wimg + 31) / 32;
  const int K = NQ + D + 1;   // chunks per strip: the last lane reaches column 32(NQ+1)-1
  const uint32_t ep32 = (uint32_t)p.epoch;
  const uint8_t* img0 = static_cast<const uint8_t*>(p.grid);
  uint8_t* out0 = static_cast<uint8_t*>(p.table);

  for (int i = threadIdx.x; i < W * kAdRing * 32; i += blockDim.x) (&ring[0][0][0])[i] = 0ull;
  if (threadIdx.x < W) cons[threadIdx.x] = 0;
  __syncthreads();

  uint32_t iter = 0;
  while (true) {
    if (threadIdx.x == 0) {
      int s = (int)atomicAdd(&ctl->claim, 1u);
      if (ld_volatile_u32(&ctl->abort)) s = INT_MAX;
      strip_sh = s;
    }
    __syncthreads();
    // batched FS: claim q -> (strip q / B, image q % B), strip-major, so the B images' strip
    // pipelines advance together; image b = rows [b H, (b+1) H) of the grid / table
    const int B = p.batch > 1 ? p.batch : 1;
    const int q = strip_sh;
    if (q >= p.nstrips * B) break;
    const int s = q / B, bimg = q - s * B;
    const int64_t row0 = (int64_t)s * SH + (wid * 32 + lane) * R;
    const uint8_t* img = img0 + (int64_t)bimg * H * p.grid_pitch;
    uint8_t* out = out0 + (int64_t)bimg * H * p.table_pitch;
    bool rvalid[R];
    const uint8_t* rin[R];
    uint8_t* rout[R];
    uint32_t inbase[R];
    int nq[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      rvalid[r] = row0 + r < H;
      rin[r] = img + (rvalid[r] ? row0 + r : 0) * p.grid_pitch;
      rout[r] = out + (rvalid[r] ? row0 + r : 0) * p.table_pitch;
      inbase[r] = smem_u32(&inr[wid][lane][r][0][0]);
      nq[r] = (-OFS - D * lane - 2 * r) >> 4;   // floor(first column / 16)
    }
    const uint32_t base = iter * (uint32_t)NQ + 1u;

    // ---- input prologue: kFsAhead chunks per row from the row's first column
    for (int a = 0; a < kFsAhead; ++a) {
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const bool in = rvalid[r] && nq[r] >= 0 && 16 * nq[r] < Wimg;
        fs_cp16(inbase[r] + (nq[r] & (kFsIn - 1)) * 16, rin[r] + (in ? 16 * nq[r] : 0), in ? 16u : 0u);
        ++nq[r];
      }
      cp_async_commit();
    }
    cp_async_wait_group<kFsAhead - 4>();
    __syncwarp();
    // inputs of the first 8 steps (the step loop loads the NEXT group's inputs one group ahead:
    // LDS.U8 + I2F on the pixel chain cost ~40 cycles per step)
    float inq[R][8];
#pragma unroll
    for (int r = 0; r < R; ++r)
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int c = -OFS + u - D * lane - 2 * r;
        inq[r][u] = fs_u8f(inr[wid][lane][r][(c >> 4) & (kFsIn - 1)][c & 15]);
      }

    // ---- links (the adiag protocol)
    const int topsrc = (wid > 0) ? 1 : (s > 0 ? 2 : 0);
    const bool last_strip = (s == p.nstrips - 1);
    const int botsnk = (wid < W - 1) ? 1 : (last_strip ? 0 : 2);
    uint64_t* ring_top = &ring[wid][0][0];
    uint64_t* ring_bot = &ring[(wid + 1) % W][0][0];
    const int64_t brow = (int64_t)bimg * p.nstrips + s;   // this strip's boundary row (per image)
    const uint64_t* gprev = static_cast<const uint64_t*>(p.bnd) + (brow - 1) * p.bnd_stride;
    uint64_t* gmine = static_cast<uint64_t*>(p.bnd) + brow * p.bnd_stride;
    uint64_t tp = 0, tq1 = (topsrc == 2) ? ad_ld_gpu(gprev + lane) : 0ull;

    float fifo[E + 3];
#pragma unroll
    for (int d = 0; d < E + 3; ++d) fifo[d] = 0.0f;
    float h[R][3];   // h[r][d]: row r's error at step tau-1-d (L of row r, UR/U/UL of row r+1)
#pragma unroll
    for (int r = 0; r < R; ++r) h[r][0] = h[r][1] = h[r][2] = 0.0f;
    bool ok = true;

    for (int k = 0; k < K && ok; ++k) {
      // publish bottom chunk k-1-D (staged by lane 31 during chunk k-1)
      const int j = k - 1 - D;
      if (botsnk != 0 && j >= 0 && j < NQ) {
        __syncwarp();
        const float v = stg[wid][lane];
        __syncwarp();
        if (botsnk == 1) {
          const uint32_t tag = base + (uint32_t)j;
          if (j >= kAdRing) {
            Backoff bo;
            while ((int)((uint32_t)ad_ld_smem_i32(&cons[wid + 1]) - (tag - kAdRing)) < 0)
              if (!bo.tick(ctl, p.timeout_ns)) { ok = false; break; }
          }
          uint64_t* d = ring_bot + (j & (kAdRing - 1)) * 32 + lane;
          asm volatile("st.volatile.shared.u64 [%0], %1;" ::"r"(smem_u32(d)), "l"(ad_pair(ad_bits(v), tag)) : "memory");
        } else {
          uint64_t* d = gmine + 32 * (int64_t)j + lane;
          asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(d), "l"(ad_pair(ad_bits(v), ep32)) : "memory");
        }
      }
      if (!__all_sync(0xffffffffu, ok)) { ok = false; break; }
      // acquire top chunk k (columns 32k + lane)
      if (k < NQ) {
        if (topsrc == 0) {
          tp = 0ull;   // row -1: errors 0
        } else {
          const uint64_t* src;
          uint32_t tag;
          if (topsrc == 1) {
            src = ring_top + (k % kAdRing) * 32 + lane;
            tag = base + (uint32_t)k;
            tp = ad_ld_smem(src);
          } else {
            src = gprev + 32 * (int64_t)k + lane;
            tag = ep32;
            tp = tq1;   // loaded half a chunk ago (group 2 of the previous chunk)
          }
          if (!__all_sync(0xffffffffu, (uint32_t)(tp >> 32) == tag)) {
            Backoff bo;
            int spins = 0;
            while (true) {
              if ((uint32_t)(tp >> 32) != tag) tp = (topsrc == 1) ? ad_ld_smem(src) : ad_ld_gpu(src);
              if (__all_sync(0xffffffffu, (uint32_t)(tp >> 32) == tag)) break;
              if (++spins > p.spin_polls && !bo.tick(ctl, p.timeout_ns)) { ok = false; break; }
            }
            if (!__all_sync(0xffffffffu, ok)) { ok = false; break; }
          }
          if (topsrc == 1 && lane == 0) ad_st_smem_i32(&cons[wid], (int)(base + (uint32_t)k));
        }
      } else {
        tp = 0ull;   // columns >= n: injected values never reach a stored pixel
      }
      // chunk k's top row -> shared memory; lane 31 reads its 8 injections per group with two
      // broadcast LDS.128 one group ahead (a per-step SHFL was scheduled late by ptxas)
      __syncwarp();
      tstg[wid][lane] = ad_val<float>(tp);
      __syncwarp();
      float injq[8];
      {
        const float4 a0 = reinterpret_cast<const float4*>(&tstg[wid][0])[0];
        const float4 a1 = reinterpret_cast<const float4*>(&tstg[wid][0])[1];
        injq[0] = a0.x; injq[1] = a0.y; injq[2] = a0.z; injq[3] = a0.w;
        injq[4] = a1.x; injq[5] = a1.y; injq[6] = a1.z; injq[7] = a1.w;
      }

      // ---- 32 steps: tau = 32k - OFS + su (fully unrolled: the period test below is static)
#pragma unroll
      for (int g = 0; g < 4; ++g) {
        // the next chunk's strip-boundary pair, half a chunk ahead: late enough that the producer
        // has usually published it (a stale pair is caught by the tag check and re-polled)
        if (g == LDDP_FSK_PG && topsrc == 2 && k + 1 < NQ)
          tq1 = ad_ld_gpu_pf(reinterpret_cast<const uint64_t*>(gprev) + 32 * (k + 1) + lane);   // relaxed.gpu: races the pair store
        float bv[8];
        float inn[R][8], injn[8];
        if (g < 3) {
          const float4 a0 = reinterpret_cast<const float4*>(&tstg[wid][8 * g + 8])[0];
          const float4 a1 = reinterpret_cast<const float4*>(&tstg[wid][8 * g + 8])[1];
          injn[0] = a0.x; injn[1] = a0.y; injn[2] = a0.z; injn[3] = a0.w;
          injn[4] = a1.x; injn[5] = a1.y; injn[6] = a1.z; injn[7] = a1.w;
        }
#pragma unroll
        for (int r = 0; r < R; ++r)
#pragma unroll
          for (int u = 0; u < 8; ++u) {
            const int cn = 32 * k - OFS + 8 * g + 8 + u - D * lane - 2 * r;
            inn[r][u] = fs_u8f(inr[wid][lane][r][(cn >> 4) & (kFsIn - 1)][cn & 15]);
          }
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const int tau = 32 * k - OFS + 8 * g + u;
          float e[R];
#pragma unroll
          for (int r = 0; r < R; ++r) {
            const int c = tau - D * lane - 2 * r;
            const float UR = r == 0 ? fifo[E] : h[r - 1][0];
            const float U = r == 0 ? fifo[E + 1] : h[r - 1][1];
            const float UL = r == 0 ? fifo[E + 2] : h[r - 1][2];
            uint8_t o;
            float x = F::f(h[r][0], UL, U, UR, 0, 0, inq[r][u], 0, 0, 0, o);
            e[r] = ((unsigned)c < (unsigned)Wimg) ? x : 0.0f;   // columns -1 and W are errors 0
            outr[wid][lane][r][(c >> 4) & (kFsOut - 1)][c & 15] = o;
          }
#pragma unroll
          for (int r = 0; r < R; ++r) {
            h[r][2] = h[r][1];
            h[r][1] = h[r][0];
            h[r][0] = e[r];
          }
          bv[u] = e[R - 1];
          const float inj = injq[u];
          const float sv = (lane == 31) ? inj : e[R - 1];
          const float rv = __shfl_sync(0xffffffffu, sv, (lane + 31) & 31);
#pragma unroll
          for (int d = E + 2; d > 0; --d) fifo[d] = fifo[d - 1];
          fifo[0] = rv;
          if ((tau & 15) == 15) {
            // period end: per row, flush the completed output chunk and issue the next input chunk
#pragma unroll
            for (int r = 0; r < R; ++r) {
              const int c = tau - D * lane - 2 * r;
              const int qd = ((c + 1) >> 4) - 1;
              if (rvalid[r] && qd >= 0 && 16 * qd < Wimg) {
                const uint4 w4 = *reinterpret_cast<const uint4*>(&outr[wid][lane][r][qd & (kFsOut - 1)][0]);
                *reinterpret_cast<uint4*>(rout[r] + 16 * qd) = w4;
              }
              const bool in2 = rvalid[r] && nq[r] >= 0 && 16 * nq[r] < Wimg;
              fs_cp16(inbase[r] + (nq[r] & (kFsIn - 1)) * 16, rin[r] + (in2 ? 16 * nq[r] : 0), in2 ? 16u : 0u);
              ++nq[r];
            }
            cp_async_commit();
            cp_async_wait_group<kFsAhead - 4>();
            __syncwarp();
          }
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) {
#pragma unroll
          for (int r = 0; r < R; ++r) inq[r][u] = inn[r][u];
          if (g < 3) injq[u] = injn[u];
        }
        if (lane == 31) {
          uint4* d = reinterpret_cast<uint4*>(&stg[wid][8 * g]);
          d[0] = make_uint4(ad_bits(bv[0]), ad_bits(bv[1]), ad_bits(bv[2]), ad_bits(bv[3]));
          d[1] = make_uint4(ad_bits(bv[4]), ad_bits(bv[5]), ad_bits(bv[6]), ad_bits(bv[7]));
        }
      }
    }
    // the last staged bottom chunk (K - 1 - D)
    if (ok && botsnk != 0) {
      const int j = K - 1 - D;
      if (j >= 0 && j < NQ) {
        __syncwarp();
        const float v = stg[wid][lane];
        __syncwarp();
        if (botsnk == 1) {
          const uint32_t tag = base + (uint32_t)j;
          if (j >= kAdRing) {
            Backoff bo;
            while ((int)((uint32_t)ad_ld_smem_i32(&cons[wid + 1]) - (tag - kAdRing)) < 0)
              if (!bo.tick(ctl, p.timeout_ns)) break;
          }
          uint64_t* d = ring_bot + (j & (kAdRing - 1)) * 32 + lane;
          asm volatile("st.volatile.shared.u64 [%0], %1;" ::"r"(smem_u32(d)), "l"(ad_pair(ad_bits(v), tag)) : "memory");
        } else {
          uint64_t* d = gmine + 32 * (int64_t)j + lane;
          asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(d), "l"(ad_pair(ad_bits(v), ep32)) : "memory");
        }
      }
    }
    cp_async_wait_group<0>();
    __syncthreads();
    ++iter;
  }
  if (threadIdx.x == 0) {
    __threadfence();
    const unsigned d = atomicAdd(&ctl->done, 1u);
    if (d == gridDim.x - 1) {
      atomicExch(&ctl->claim, 0u);
      atomicExch(&ctl->done, 0u);
    }
  }
}

// W warps per CTA (strip = 32 W R rows), E = extra lane lag, R rows per lane.  grid <= strips.
cudaError_t launch_fsk(const FillParams& p, int W, int E, int R, int grid, cudaStream_t s) {
#define LDDP_FSK(w, e, r)                                                \
  if (W == w && E == e && R == r) {                                      \
    fsk_kernel<w, e, r><<<grid, w * 32, 0, s>>>(p);                      \
    return cudaGetLastError();                                           \
  }
  // default (1, 1, 1); the others are the measured alternatives kept for sweeps
  LDDP_FSK(1, 1, 1) LDDP_FSK(1, 0, 1) LDDP_FSK(1, 2, 1) LDDP_FSK(1, 1, 2) LDDP_FSK(1, 0, 2) LDDP_FSK(4, 1, 1)
  LDDP_FSK(2, 1, 1)
#undef LDDP_FSK
  return cudaErrorInvalidValue;
}

}  // namespace lddp
