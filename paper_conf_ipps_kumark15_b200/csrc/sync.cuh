// sync.cuh -- device synchronisation primitives of the persistent LDDP kernels (sm_100a).
//
// * mbarrier producer/consumer rings between warps of one CTA (intra-strip handoff);
// * epoch-tagged release/acquire progress flags in global memory between CTAs (strip handoff,
//   SURVEY §8(a3)) and between GPUs over NVLink (system scope, §8(e));
// * a watchdog: every dependency wait is bounded (globaltimer), so a protocol bug reports
//   LDDP_ERR_TIMEOUT through the workspace status word instead of hanging the device.
#pragma once
#include <cstdint>

namespace lddp {

struct Control {                 // workspace header (device), zeroed by lddp_workspace_init
  unsigned int claim;            // next strip / band to claim (persistent scheduler)
  unsigned int done;             // CTAs finished (last one resets claim / done)
  unsigned int status;           // 0 or lddp_status of a device-side failure
  unsigned int abort;            // set on watchdog expiry: every wait gives up
  unsigned int pad[12];
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
// TMA bulk copy global -> shared, completion signalled on an mbarrier (complete_tx bytes).
// dst / src 16-byte aligned, bytes a multiple of 16.
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
// Order this thread's prior generic-proxy shared-memory accesses before later async-proxy
// (TMA) writes to the same buffer.
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// Ampere-style per-thread async copy global -> shared (LDGSTS); src_bytes 0 zero-fills.
__device__ __forceinline__ void cp_async_8(void* dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(smem_u32(dst)), "l"(src), "r"(src_bytes)
               : "memory");
}
__device__ __forceinline__ void cp_async_4(void* dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(smem_u32(dst)), "l"(src), "r"(src_bytes)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait_group() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

__device__ __forceinline__ uint64_t globaltimer_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ uint64_t ld_acquire_gpu(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_relaxed_gpu(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
__device__ __forceinline__ void st_release_gpu(uint64_t* p, uint64_t v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_release_sys(uint64_t* p, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned ld_volatile_u32(const unsigned* p) {
  return *reinterpret_cast<const volatile unsigned*>(p);
}

// Watchdog bookkeeping for one waiting thread.
// kSleep: back off with __nanosleep between polls of a global flag (spares L2 bandwidth);
// mbarrier waits do not sleep (try_wait already suspends the warp in hardware until the
// phase flips or a short time limit expires).
template <bool kSleep = true>
struct Watch {
  uint64_t t0;
  uint32_t spins;
  __device__ __forceinline__ Watch() : t0(0), spins(0) {}
  // Returns false if the wait must be abandoned (abort flag or timeout).
  __device__ __forceinline__ bool tick(Control* ctl, uint64_t timeout_ns) {
    ++spins;
    if (kSleep) {
      if (spins < 64) return true;
      __nanosleep(spins < 4096 ? 20 : 200);
    }
    if ((spins & 1023) != 0) return true;
    if (ld_volatile_u32(&ctl->abort)) return false;
    uint64_t now = globaltimer_ns();
    if (t0 == 0) { t0 = now; return true; }
    if (now - t0 > timeout_ns) {
      atomicCAS(&ctl->status, 0u, 8u /* LDDP_ERR_TIMEOUT */);
      atomicExch(&ctl->abort, 1u);
      return false;
    }
    return true;
  }
};

// Polling wait with an early back-off: a consumer warp spinning on shared / global memory
// competes with the producer warps of its SM for the MIO / LSU pipes (SHFL, LDS), so after a
// couple of failed polls it sleeps between polls.
struct Backoff {
  uint64_t t0;
  uint32_t spins;
  __device__ __forceinline__ Backoff() : t0(0), spins(0) {}
  __device__ __forceinline__ bool tick(Control* ctl, uint64_t timeout_ns) {
    ++spins;
    if (spins >= 2) __nanosleep(spins < 256 ? 32 : 256);
    if ((spins & 255) != 0) return true;
    if (ld_volatile_u32(&ctl->abort)) return false;
    uint64_t now = globaltimer_ns();
    if (t0 == 0) { t0 = now; return true; }
    if (now - t0 > timeout_ns) {
      atomicCAS(&ctl->status, 0u, 8u /* LDDP_ERR_TIMEOUT */);
      atomicExch(&ctl->abort, 1u);
      return false;
    }
    return true;
  }
};

// Wait until an epoch-tagged flag (epoch << 32 | count) reaches `target`.
template <bool kSys>
__device__ __forceinline__ bool wait_flag(const uint64_t* flag, uint64_t target, Control* ctl,
                                          uint64_t timeout_ns) {
  Watch<true> w;
  while (true) {
    uint64_t v = kSys ? ld_acquire_sys(flag) : ld_acquire_gpu(flag);
    if (v >= target) return true;
    if (!w.tick(ctl, timeout_ns)) return false;
  }
}

// Wait until an epoch-tagged flag EQUALS `target` (multi-GPU window slots are reused every
// other fill: an older epoch must not pass).
__device__ __forceinline__ bool wait_flag_eq_sys(const uint64_t* flag, uint64_t target, Control* ctl,
                                                 uint64_t timeout_ns) {
  Watch<true> w;
  while (true) {
    if (ld_acquire_sys(flag) == target) return true;
    if (!w.tick(ctl, timeout_ns)) return false;
  }
}

// ---- multi-GPU receive window protocol (lddp.h "multi-GPU column strips"); wepoch = fill k
// Consumer, before reading strip s's left column (rows top_s - 1 .. top_s + SH - 1): the strip's
// flag and the previous strip's (its last row) must carry this fill's epoch.
template <class Params>
__device__ __forceinline__ bool window_consume_wait(const Params& p, int s, Control* ctl) {
  const uint64_t tag = (p.wepoch << 32) | 1u;
  if (!wait_flag_eq_sys(p.lflag_in + s, tag, ctl, p.timeout_ns)) return false;
  return s == 0 || wait_flag_eq_sys(p.lflag_in + s - 1, tag, ctl, p.timeout_ns);
}
// Consumer, after every thread of the strip has read its left values (caller synchronises):
// tell rank g-1 that slot (k & 1) of strip s may be reused.
template <class Params>
__device__ __forceinline__ void window_consume_ack(const Params& p, int s) {
  if (p.ack_out != nullptr) st_release_sys(p.ack_out + s, p.wepoch);
}
// Producer, before storing strip s's right column into rank g+1's slot (k & 1): rank g+1 has
// finished reading fill k-2 there (strips s and s+1, which reads strip s's last row).
template <class Params>
__device__ __forceinline__ bool window_produce_wait(const Params& p, int s, Control* ctl) {
  if (p.wepoch <= 2) return true;
  const uint64_t need = p.wepoch - 2;
  for (int t = s; t <= s + 1 && t < p.nstrips; ++t) {
    Watch<true> w;
    while (ld_acquire_sys(p.ack_in + t) < need)
      if (!w.tick(ctl, p.timeout_ns)) return false;
  }
  return true;
}

// Acquire pattern without an L1 invalidation per poll: relaxed polls, then one acq_rel fence
// once the released value is observed.  Returns the observed flag in `seen`.
__device__ __forceinline__ bool wait_flag_relaxed(const uint64_t* flag, uint64_t target, Control* ctl,
                                                  uint64_t timeout_ns, uint64_t& seen) {
  Watch<true> w;
  while (true) {
    uint64_t v = ld_relaxed_gpu(flag);
    if (v >= target) {
      seen = v;
      fence_acq_rel_gpu();
      return true;
    }
    if (!w.tick(ctl, timeout_ns)) return false;
  }
}

// Bounded mbarrier wait (phase parity).
__device__ __forceinline__ bool mbar_wait(uint64_t* bar, uint32_t parity, Control* ctl,
                                          uint64_t timeout_ns) {
  if (mbar_try_wait(bar, parity)) return true;
  Watch<false> w;
  while (!mbar_try_wait(bar, parity)) {
    if (!w.tick(ctl, timeout_ns)) return false;
  }
  return true;
}

}  // namespace lddp
