// Inline-PTX helpers for the sm_100a tcgen05 / TMA / mbarrier kernels.
#pragma once

#include <cuda_bf16.h>
#include <cstdint>

#ifndef TEMCO_SUSPEND_HINT_NS
#define TEMCO_SUSPEND_HINT_NS 1000000
#endif

namespace temco {
namespace ptx {


__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// one arrive per warp: the warp's prior memory / tcgen05 operations are ordered
// by __syncwarp, then lane 0 arrives (barrier counts are in warps, not threads:
// 256 single-thread arrives on one mbarrier serialise for thousands of cycles)
__device__ __forceinline__ void warp_arrive(uint64_t* bar) {
  __syncwarp();
  if ((threadIdx.x & 31) == 0) mbar_arrive(bar);
}

__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
      "selp.u32 %0, 1, 0, p;\n"
      "}\n"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}

// Wait for the phase with the given parity.  Watchdog: a wait that has not
// completed after ~4 s (a protocol bug) traps, turning a hung kernel into a
// launch error instead of a wedged GPU.
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  if (mbar_try_wait(bar, parity)) return;
  const long long t0 = clock64();
  for (uint32_t n = 1;; ++n) {
    if (mbar_try_wait(bar, parity)) return;
    if ((n & 1023u) == 0 && clock64() - t0 > 8000000000LL) __trap();
  }
}

// same, with a suspend-time hint: the waiting warp sleeps until the phase
// completes (or the hint expires) instead of re-issuing try_wait, leaving the
// SM sub-partition's issue slots to the single-thread producer / MMA roles
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity), "r"(TEMCO_SUSPEND_HINT_NS)
      : "memory");
}

__device__ __forceinline__ void tma_load_2d(void* dst, const void* map, uint64_t* bar, int x, int y) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
          smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(x), "r"(y)
      : "memory");
}

// K-major, 128-byte swizzle UMMA shared-memory descriptor (8-row groups 1024 B apart)
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr) {
  return (uint64_t)((saddr & 0x3FFFF) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}

// K-major descriptor for a K atom of `aw` bf16 elements per row (16, 32 or 64):
// swizzle = row bytes (SW32 / SW64 / SW128), 8-row groups 8 * row bytes apart.
// The atom base must be aligned to 8 * row bytes.
__device__ __forceinline__ uint64_t umma_desc_k(uint32_t saddr, int aw) {
  const uint64_t layout = aw == 64 ? 2 : aw == 32 ? 4 : 6;
  const uint64_t sbo = (uint64_t)(16 * aw) >> 4;
  return (uint64_t)((saddr & 0x3FFFF) >> 4) | ((uint64_t)1 << 16) | (sbo << 32) | ((uint64_t)1 << 46) |
         (layout << 61);
}

// physical 16-byte chunk of logical chunk k in row r of a K atom with `aw` elements
__host__ __device__ __forceinline__ int swz_chunk(int r, int k, int aw) {
  return aw == 64 ? (k ^ (r & 7)) : aw == 32 ? (k ^ ((r >> 1) & 3)) : (k ^ ((r >> 2) & 1));
}

// kind::f16 instruction descriptor: bf16 A/B, fp32 D, K-major A/B
__host__ __device__ constexpr uint32_t idesc_bf16(int M, int N) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

__device__ __forceinline__ void mma_bf16(uint32_t dtmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(dtmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc));
}

__device__ __forceinline__ void mma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
               : "memory");
}

// warp-wide variants: the whole (converged) warp executes, one elected lane issues
__device__ __forceinline__ void mma_bf16_w(uint32_t dtmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n"
      ".reg .pred p, e;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(dtmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc));
}

__device__ __forceinline__ void mma_commit_w(uint64_t* bar) {
  asm volatile(
      "{\n"
      ".reg .pred e;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n"
      "}\n" ::"r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ void mbar_expect_tx_w(uint64_t* bar, uint32_t bytes) {
  asm volatile(
      "{\n"
      ".reg .pred e;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "@e mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(bytes)
      : "memory");
}

__device__ __forceinline__ void tma_load_2d_w(void* dst, const void* map, uint64_t* bar, int x, int y) {
  asm volatile(
      "{\n"
      ".reg .pred e;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "@e cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];\n"
      "}\n" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(x), "r"(y)
      : "memory");
}

__device__ __forceinline__ void tma_load_4d_w(void* dst, const void* map, uint64_t* bar, int c, int w, int h, int n) {
  asm volatile(
      "{\n"
      ".reg .pred e;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "@e cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2];\n"
      "}\n" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c), "r"(w), "r"(h), "r"(n)
      : "memory");
}

__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

#define TMEM_REGS32(v)                                                                                            \
  "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), "=r"(v[8]),       \
      "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]), "=r"(v[16]),        \
      "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]), "=r"(v[24]),       \
      "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&v)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, "
      "%16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
      : TMEM_REGS32(v)
      : "r"(taddr));
}

__device__ __forceinline__ void tmem_st32(uint32_t taddr, const uint32_t (&v)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
      "%15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31, %32};" ::"r"(taddr),
      "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]), "r"(v[9]),
      "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15]), "r"(v[16]), "r"(v[17]), "r"(v[18]),
      "r"(v[19]), "r"(v[20]), "r"(v[21]), "r"(v[22]), "r"(v[23]), "r"(v[24]), "r"(v[25]), "r"(v[26]), "r"(v[27]),
      "r"(v[28]), "r"(v[29]), "r"(v[30]), "r"(v[31])
      : "memory");
}

__device__ __forceinline__ void tmem_ld8(uint32_t taddr, uint32_t (&v)[8]) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
               : "r"(taddr));
}

__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

__device__ __forceinline__ uint32_t pack_bf16(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}

// silu(x) = h + h tanh(h), h = x / 2, one MUFU operation (tanh.approx.f32, relative error
// ~2^-11) instead of an exponential and a reciprocal: bf16-output tensor-core epilogues only
__device__ __forceinline__ float silu_fast(float x) {
  const float h = 0.5f * x;
  float t;
  asm("tanh.approx.f32 %0, %1;" : "=f"(t) : "f"(h));
  return fmaf(h, t, h);
}

// bf16x2 of (silu(a), silu(b)) for epilogues whose output is bf16: silu(x) = h + h tanh(h),
// h = x / 2, with one packed bf16x2 tanh (one MUFU operation per two values instead of an
// exponential and a reciprocal per value); tanh in bf16 adds <= 2^-9 |h| absolute error, below
// the bf16 rounding of the output itself
__device__ __forceinline__ uint32_t pack_silu_bf16(float a, float b) {
  const float ha = 0.5f * a, hb = 0.5f * b;
  uint32_t hp = pack_bf16(ha, hb), th;
  asm("tanh.approx.bf16x2 %0, %1;" : "=r"(th) : "r"(hp));
  const float ta = __uint_as_float(th << 16), tb = __uint_as_float(th & 0xFFFF0000u);
  return pack_bf16(fmaf(ha, ta, ha), fmaf(hb, tb, hb));
}

// bf16x2 of (max(a, 0), max(b, 0)) in one instruction
__device__ __forceinline__ uint32_t pack_bf16_relu(float a, float b) {
  uint32_t r;
  asm("cvt.rn.relu.bf16x2.f32 %0, %2, %1;" : "=r"(r) : "f"(a), "f"(b));
  return r;
}

// 4D tiled TMA load (NHWC box: channels, w, h, n); out-of-range coordinates zero-fill
__device__ __forceinline__ void tma_load_4d(void* dst, const void* map, uint64_t* bar, int c, int w, int h, int n) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], "
      "[%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c), "r"(w), "r"(h), "r"(n)
      : "memory");
}

// asynchronous 16-byte global->shared copy; src_bytes = 0 zero-fills (padding)
__device__ __forceinline__ void cp_async16(void* dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(dst)), "l"(src), "r"(src_bytes)
               : "memory");
}

// arrive on `bar` once all prior cp.async of this thread have completed
__device__ __forceinline__ void cp_async_arrive(uint64_t* bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }


// ---------------------------------------------------------------------------
// 2-CTA cluster (cta_group::2) helpers
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}

// shared::cluster address of the same shared variable in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t mapa_shared(uint32_t saddr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
  return r;
}

__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

__device__ __forceinline__ void fence_mbar_init_cluster() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

// arrive on an mbarrier given by its shared::cluster address (possibly the peer CTA's).
// Default semantics (release at CTA scope): a bare SYNCS arrive -- .release.cluster
// compiles to MEMBAR.ALL.GPU (~1000 cycles).  The data the arrivals publish is
// tcgen05 state (ordered by tcgen05.fence::before_thread_sync) or shared memory
// handed to the async proxy (fence.proxy.async), as in CUTLASS's 2-SM pipelines.
__device__ __forceinline__ void mbar_arrive_cluster(uint32_t caddr) {
  asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(caddr) : "memory");
}

// one arrive per warp on a (possibly remote) barrier, after the warp's prior work
__device__ __forceinline__ void warp_arrive_cluster(uint32_t caddr) {
  __syncwarp();
  if ((threadIdx.x & 31) == 0) mbar_arrive_cluster(caddr);
}

__device__ __forceinline__ bool mbar_try_wait_cluster(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
      "selp.u32 %0, 1, 0, p;\n"
      "}\n"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}

// wait for a phase whose arrivals come from the peer CTA too (default acquire.cta:
// .acquire.cluster adds an L1 invalidate per wake-up); watchdog as mbar_wait
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t parity) {
  if (mbar_try_wait_cluster(bar, parity)) return;
  const long long t0 = clock64();
  for (uint32_t n = 1;; ++n) {
    if (mbar_try_wait_cluster(bar, parity)) return;
    if ((n & 1023u) == 0 && clock64() - t0 > 8000000000LL) __trap();
  }
}

// 2D TMA load issued by either CTA of a pair; completion bytes go to the barrier at
// shared::cluster address `bar_c` (the leader CTA's), data to this CTA's `dst`
__device__ __forceinline__ void tma_load_2d_pair(void* dst, const void* map, uint32_t bar_c, int x, int y) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], "
      "[%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(bar_c), "r"(x), "r"(y)
      : "memory");
}

// Wait with the spin loop (and the ~4 s watchdog) inside the asm: no data-dependent
// branch at C level, so the compiler keeps the caller's loop state warp-uniform (uniform
// registers feeding tcgen05.mma directly instead of per-instruction broadcasts).
__device__ __forceinline__ void mbar_wait_u(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p, q;\n"
      ".reg .u64 t0, t1;\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@p bra DONE_%=;\n"
      "mov.u64 t0, %%clock64;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@p bra DONE_%=;\n"
      "mov.u64 t1, %%clock64;\n"
      "sub.u64 t1, t1, t0;\n"
      "setp.gt.u64 q, t1, 8000000000;\n"
      "@q trap;\n"
      "bra WAIT_%=;\n"
      "DONE_%=:\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// single-thread forms (the caller is one lane; no elect)
__device__ __forceinline__ void mma2_bf16(uint32_t dtmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(dtmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc));
}

__device__ __forceinline__ void mma2_commit_mc(uint64_t* bar, uint16_t mask) {
  asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
                   smem_u32(bar)),
               "h"(mask)
               : "memory");
}

// warp-wide: one elected lane issues a cta_group::2 MMA (leader CTA only)
__device__ __forceinline__ void mma2_bf16_w(uint32_t dtmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n"
      ".reg .pred p, e;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(dtmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc));
}

__device__ __forceinline__ uint4 lds128(uint32_t saddr) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(saddr));
  return v;
}

// UMMA shared-memory descriptor halves (K-major, swizzle by K atom width aw = 64 / 32 / 16
// elements: SW128 / SW64 / SW32): lo = start address >> 4 | LBO 1, hi = SBO | version | layout.
// Advancing K by 16 elements adds 2 to lo.
__host__ __device__ __forceinline__ uint32_t udesc_lo(uint32_t saddr) { return ((saddr & 0x3FFFFu) >> 4) | 0x10000u; }
__host__ __device__ __forceinline__ uint32_t udesc_hi(int aw) {
  const uint32_t layout = aw == 64 ? 2u : aw == 32 ? 4u : 6u;
  return ((uint32_t)(16 * aw) >> 4) | (1u << 14) | (layout << 29);
}

// warp-wide: one elected lane issues nk (1..4) cta_group::2 MMAs of consecutive K16 steps
// (A, B descriptors advance by 32 bytes), the first with accumulate = acc0, the rest
// accumulating -- one asm block, so the descriptors are moved to uniform registers once
__device__ __forceinline__ void mma2_k4_w(uint32_t dtmem, uint32_t a_lo, uint32_t a_hi, uint32_t b_lo, uint32_t b_hi,
                                          uint32_t idesc, uint32_t acc0, uint32_t nk) {
  asm volatile(
      "{\n"
      ".reg .pred e, pa, pt, q1, q2, q3;\n"
      ".reg .b64 da, db;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "setp.ne.b32 pa, %6, 0;\n"
      "setp.eq.b32 pt, %7, %7;\n"
      "setp.gt.u32 q1, %7, 1;\n"
      "setp.gt.u32 q2, %7, 2;\n"
      "setp.gt.u32 q3, %7, 3;\n"
      "and.pred q1, q1, e;\n"
      "and.pred q2, q2, e;\n"
      "and.pred q3, q3, e;\n"
      "mov.b64 da, {%1, %2};\n"
      "mov.b64 db, {%3, %4};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], da, db, %5, pa;\n"
      "add.s64 da, da, 2;\n"
      "add.s64 db, db, 2;\n"
      "@q1 tcgen05.mma.cta_group::2.kind::f16 [%0], da, db, %5, pt;\n"
      "add.s64 da, da, 2;\n"
      "add.s64 db, db, 2;\n"
      "@q2 tcgen05.mma.cta_group::2.kind::f16 [%0], da, db, %5, pt;\n"
      "add.s64 da, da, 2;\n"
      "add.s64 db, db, 2;\n"
      "@q3 tcgen05.mma.cta_group::2.kind::f16 [%0], da, db, %5, pt;\n"
      "}\n" ::"r"(dtmem),
      "r"(a_lo), "r"(a_hi), "r"(b_lo), "r"(b_hi), "r"(idesc), "r"(acc0), "r"(nk));
}

// warp-wide: commit to two barriers (n = 1 or 2) in one asm block (one elect)
__device__ __forceinline__ void mma2_commit2_mc_w(uint32_t bar0, uint32_t bar1, uint32_t n) {
  asm volatile(
      "{\n"
      ".reg .pred e, e1;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "setp.gt.u32 e1, %2, 1;\n"
      "and.pred e1, e1, e;\n"
      "@e tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %3;\n"
      "@e1 tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%1], %3;\n"
      "}\n" ::"r"(bar0),
      "r"(bar1), "r"(n), "h"((uint16_t)3)
      : "memory");
}

// warp-wide: 8 K16 MMAs of two consecutive 64-wide K atoms (A atom 2 at +a2 bytes, B atom 2 at
// +b2 bytes from atom 1), one elect; the first accumulates iff acc0
__device__ __forceinline__ void mma2_k8_w(uint32_t dtmem, uint32_t a_lo, uint32_t a_hi, uint32_t b_lo, uint32_t b_hi,
                                          uint32_t a2, uint32_t b2, uint32_t idesc, uint32_t acc0) {
  asm volatile(
      "{\n"
      ".reg .pred e, pa, pt;\n"
      ".reg .b64 da, db, da2, db2;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "setp.ne.b32 pa, %8, 0;\n"
      "setp.eq.b32 pt, %5, %5;\n"
      "mov.b64 da, {%1, %2};\n"
      "mov.b64 db, {%3, %4};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], da, db, %5, pa;\n"
      "add.s64 da2, da, 2;\n add.s64 db2, db, 2;\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], da2, db2, %5, pt;\n"
      "add.s64 da2, da, 4;\n add.s64 db2, db, 4;\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], da2, db2, %5, pt;\n"
      "add.s64 da2, da, 6;\n add.s64 db2, db, 6;\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], da2, db2, %5, pt;\n"
      "cvt.u64.u32 da2, %6;\n cvt.u64.u32 db2, %7;\n"
      "add.s64 da, da, da2;\n add.s64 db, db, db2;\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], da, db, %5, pt;\n"
      "add.s64 da2, da, 2;\n add.s64 db2, db, 2;\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], da2, db2, %5, pt;\n"
      "add.s64 da2, da, 4;\n add.s64 db2, db, 4;\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], da2, db2, %5, pt;\n"
      "add.s64 da2, da, 6;\n add.s64 db2, db, 6;\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], da2, db2, %5, pt;\n"
      "}\n" ::"r"(dtmem),
      "r"(a_lo), "r"(a_hi), "r"(b_lo), "r"(b_hi), "r"(idesc), "r"(a2 >> 4), "r"(b2 >> 4), "r"(acc0));
}

// warp-wide: one K atom of a level for both units of a CTA pair in one asm block (one elect):
// for unit q < nu: [bias MMA ones x C_q into D_q, accumulate off, if bia] then nk K16 MMAs
// A x B_q into D_q (A, B advance 32 bytes per step; the first accumulates iff acc0)
__device__ __forceinline__ void mma2_atom2_w(uint32_t d0, uint32_t d1, uint32_t a_lo, uint32_t a_hi, uint32_t b0_lo,
                                             uint32_t b1_lo, uint32_t c0_lo, uint32_t c1_lo, uint32_t ones_lo,
                                             uint32_t hi16, uint32_t idesc, uint32_t nk, uint32_t nu, uint32_t bia,
                                             uint32_t acc0) {
  asm volatile(
      "{\n"
      ".reg .pred e, e1, pb, pb1, pa, pt, pf, q1, q2, q3, r1, r2, r3;\n"
      ".reg .b64 da, db, dn, dc;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "setp.gt.u32 e1, %12, 1;\n"
      "and.pred e1, e1, e;\n"
      "setp.ne.b32 pb, %13, 0;\n"
      "and.pred pb, pb, e;\n"
      "and.pred pb1, pb, e1;\n"
      "setp.ne.b32 pa, %14, 0;\n"
      "setp.eq.b32 pt, %11, %11;\n"
      "setp.ne.b32 pf, %11, %11;\n"
      "setp.gt.u32 q1, %11, 1;\n"
      "setp.gt.u32 q2, %11, 2;\n"
      "setp.gt.u32 q3, %11, 3;\n"
      "and.pred r1, q1, e1;\n"
      "and.pred r2, q2, e1;\n"
      "and.pred r3, q3, e1;\n"
      "and.pred q1, q1, e;\n"
      "and.pred q2, q2, e;\n"
      "and.pred q3, q3, e;\n"
      "mov.b64 dn, {%8, %9};\n"
      "mov.b64 dc, {%6, %9};\n"
      "@pb tcgen05.mma.cta_group::2.kind::f16 [%0], dn, dc, %10, pf;\n"
      "mov.b64 da, {%2, %3};\n"
      "mov.b64 db, {%4, %3};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], da, db, %10, pa;\n"
      "add.s64 da, da, 2;\n add.s64 db, db, 2;\n"
      "@q1 tcgen05.mma.cta_group::2.kind::f16 [%0], da, db, %10, pt;\n"
      "add.s64 da, da, 2;\n add.s64 db, db, 2;\n"
      "@q2 tcgen05.mma.cta_group::2.kind::f16 [%0], da, db, %10, pt;\n"
      "add.s64 da, da, 2;\n add.s64 db, db, 2;\n"
      "@q3 tcgen05.mma.cta_group::2.kind::f16 [%0], da, db, %10, pt;\n"
      "mov.b64 dc, {%7, %9};\n"
      "@pb1 tcgen05.mma.cta_group::2.kind::f16 [%1], dn, dc, %10, pf;\n"
      "mov.b64 da, {%2, %3};\n"
      "mov.b64 db, {%5, %3};\n"
      "@e1 tcgen05.mma.cta_group::2.kind::f16 [%1], da, db, %10, pa;\n"
      "add.s64 da, da, 2;\n add.s64 db, db, 2;\n"
      "@r1 tcgen05.mma.cta_group::2.kind::f16 [%1], da, db, %10, pt;\n"
      "add.s64 da, da, 2;\n add.s64 db, db, 2;\n"
      "@r2 tcgen05.mma.cta_group::2.kind::f16 [%1], da, db, %10, pt;\n"
      "add.s64 da, da, 2;\n add.s64 db, db, 2;\n"
      "@r3 tcgen05.mma.cta_group::2.kind::f16 [%1], da, db, %10, pt;\n"
      "}\n" ::"r"(d0),
      "r"(d1), "r"(a_lo), "r"(a_hi), "r"(b0_lo), "r"(b1_lo), "r"(c0_lo), "r"(c1_lo), "r"(ones_lo), "r"(hi16),
      "r"(idesc), "r"(nk), "r"(nu), "r"(bia), "r"(acc0));
}

// warp-wide: the elected lane's prior cta_group::2 MMAs complete -> arrive on the
// barrier at this shared offset in every CTA of `mask`
__device__ __forceinline__ void mma2_commit_mc_w(uint64_t* bar, uint16_t mask) {
  asm volatile(
      "{\n"
      ".reg .pred e;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "@e tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "h"(mask)
      : "memory");
}

__device__ __forceinline__ void prefetch_tmap(const void* map) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}

}  // namespace ptx
}  // namespace temco
