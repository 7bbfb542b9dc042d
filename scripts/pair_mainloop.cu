// Microbenchmark: the CTA-pair restore GEMM main loop in isolation (B200, sm_100a).
// 74 two-CTA clusters stream r atoms [128 px x 64] (each CTA its own pixels) and weight
// atoms [N/2 x 64] through a TMA ring and issue cta_group::2 MMAs (M = 256, N, K = 16 x 4
// per stage) into one TMEM accumulator; no epilogue.  Reports TFLOP/s for
// (N, ring stages, TMA on/off, A reuse = MMAs of different weight atoms per A atom).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o pair_mainloop scripts/pair_mainloop.cu -lcuda
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_bf16.h>
#include <cstdint>
#include <cstdio>
#include <vector>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(c)); }
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t par) {
  asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(smem_u32(b)), "r"(par) : "memory");
}
__device__ __forceinline__ void expect_tx(uint64_t* b, uint32_t n) { asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(n) : "memory"); }
__device__ __forceinline__ uint32_t mapa0(uint32_t a) { uint32_t r; asm volatile("mapa.shared::cluster.u32 %0, %1, 0;" : "=r"(r) : "r"(a)); return r; }
__device__ __forceinline__ void tma2(void* dst, const void* map, uint32_t bar, int x, int y) {
  asm volatile("cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
               ::"r"(smem_u32(dst)), "l"((uint64_t)map), "r"(bar), "r"(x), "r"(y) : "memory");
}
__device__ __forceinline__ uint64_t desc(uint32_t saddr) {
  return (uint64_t)((saddr & 0x3FFFF) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) | ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__device__ __forceinline__ void mma2(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d), "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void commit_mc(uint64_t* b) {
  asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(smem_u32(b)), "h"((uint16_t)3) : "memory");
}

struct Args { CUtensorMap amap, bmap; int N, S, tma, reuse, natoms, tiles; unsigned long long* prof; int spin; };

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(576, 1) k(const __grid_constant__ Args g) {
  extern __shared__ __align__(1024) uint8_t sm_raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)sm_raw + 1023) & ~(uintptr_t)1023);
  const int slotA = 16384, slotB = g.reuse * g.N / 2 * 128, slot = slotA + slotB;
  uint64_t* full = (uint64_t*)(sm + g.S * slot);
  uint64_t* empty = full + 16;
  uint64_t* done = empty + 16;
  uint32_t* tslot = (uint32_t*)(done + 1);
  uint32_t cta; asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(cta));
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < g.S; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    mbar_init(done, 1);
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  if (w == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tbase = *tslot;
  const int pair = blockIdx.x >> 1, npairs = gridDim.x >> 1;
  const int nstage = g.tiles * g.natoms;
  if (w == 0 && lane == 0) {
    int st = 0; uint32_t ph = 0;
    for (int i = 0; i < nstage; ++i) {
      const int tile = pair + (i / g.natoms) * npairs, a = i % g.natoms;
      mbar_wait(&empty[st], ph ^ 1);
      if (cta == 0) expect_tx(&full[st], g.tma ? 2u * (uint32_t)slot : 0u);
      if (g.tma) {
        const uint32_t fb = mapa0(smem_u32(&full[st]));
        tma2(sm + st * slot, &g.amap, fb, a * 64, tile * 256 + cta * 128);
        for (int r = 0; r < g.reuse; ++r)
          tma2(sm + st * slot + slotA + r * (g.N / 2 * 128), &g.bmap, fb, a * 64, (r * 2 + cta) * (g.N / 2));
      }
      if (++st == g.S) st = 0, ph ^= 1;
    }
  } else if (w == 1 && cta == 0) {
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(g.N >> 3) << 17) | ((uint32_t)(256 >> 4) << 24);
    int st = 0; uint32_t ph = 0;
    long long tw = 0, tm = 0, tc = 0;
    const long long tstart = clock64();
    for (int i = 0; i < nstage; ++i) {
      long long a0 = clock64();
      mbar_wait(&full[st], ph);
      long long a1 = clock64();
      tw += a1 - a0;
      asm volatile("tcgen05.fence::after_thread_sync;");
      if (lane == 0) {
        const uint32_t sa = smem_u32(sm + st * slot);
        const uint64_t ad = desc(sa);
        for (int r = 0; r < g.reuse; ++r) {
          const uint64_t bd = desc(sa + slotA + r * (g.N / 2 * 128));
          const uint32_t dt = tbase + (uint32_t)((r * g.N) & 511);
          for (int kk = 0; kk < 4; ++kk) mma2(dt, ad + 2 * kk, bd + 2 * kk, idesc, (i | kk) > 0);
        }
        long long a2 = clock64();
        tm += a2 - a1;
        commit_mc(&empty[st]);
        tc += clock64() - a2;
      }
      __syncwarp();
      if (++st == g.S) st = 0, ph ^= 1;
    }
    if (lane == 0) commit_mc(done);
    if (lane == 0 && blockIdx.x == 0) {
      g.prof[0] = clock64() - tstart;
      g.prof[1] = tw;
      g.prof[2] = tm;
      g.prof[3] = tc;
    }
  }
  if (w >= 2) {
    if (g.spin == 1) mbar_wait(done, 0);   // all extra warps sleep in try_wait on `done`
    else if (w == 2) mbar_wait(done, 0);
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (w == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;");
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(tbase));
  }
}

int main() {
  PFN_cuTensorMapEncodeTiled_v12000 enc;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q);
  const int natoms = 12, ntiles = 196 * 4;   // K = 768 per tile, 4 "units" worth of tiles
  const size_t npix = (size_t)ntiles * 256, K = 64 * natoms;
  __nv_bfloat16 *A, *B;
  cudaMalloc(&A, npix * K * 2);
  cudaMalloc(&B, 512 * K * 2);
  cudaMemset(A, 0, npix * K * 2);
  cudaMemset(B, 0, 512 * K * 2);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
  unsigned long long* prof;
  cudaMalloc(&prof, 64);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  int nsm = 148;
  for (int spin : {0, 1})
  for (int N : {128, 256})
    for (int reuse : {1, 2})
      for (int S : {4})
        for (int tma : {1}) {
          if (reuse * N > 256) continue;
          Args g{};
          g.prof = prof;
          g.N = N; g.S = S; g.tma = tma; g.reuse = reuse; g.natoms = natoms; g.tiles = ntiles / (nsm / 2);
          const int slot = 16384 + reuse * N / 2 * 128;
          if (S * slot + 1024 + 512 > 227 * 1024) continue;
          cuuint64_t da[2] = {K, npix}, sa[1] = {K * 2};
          cuuint32_t ba[2] = {64, 128}, es[2] = {1, 1};
          enc(&g.amap, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, A, da, sa, ba, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
              CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
          cuuint64_t db[2] = {K, 512};
          cuuint32_t bb[2] = {64, (cuuint32_t)(N / 2)};
          enc(&g.bmap, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, B, db, sa, bb, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
              CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
          const int smem = S * slot + 2048;
          const int nthr = spin ? 576 : 128;
          g.spin = spin;
          for (int rep = 0; rep < 3; ++rep) k<<<nsm, nthr, smem>>>(g);
          cudaEventRecord(e0);
          const int it = 5;
          for (int rep = 0; rep < it; ++rep) k<<<nsm, nthr, smem>>>(g);
          cudaEventRecord(e1);
          cudaError_t err = cudaDeviceSynchronize();
          if (err != cudaSuccess) { printf("err %s\n", cudaGetErrorString(err)); return 1; }
          float ms; cudaEventElapsedTime(&ms, e0, e1); ms /= it;
          const double flops = 2.0 * (nsm / 2) * g.tiles * 256.0 * natoms * 64 * N * reuse;
          const double bytes = (double)(nsm / 2) * g.tiles * natoms * 2 * slot;
          unsigned long long pr[4];
          cudaMemcpy(pr, prof, 32, cudaMemcpyDeviceToHost);
          const double nst = (double)g.tiles * natoms;
          printf("spin=%d ", spin);
          printf("N=%3d reuse=%d S=%d tma=%d: %7.3f ms  %7.1f TFLOP/s  L2->SMEM %6.0f GB/s (%.1f B/cyc/SM @1.9GHz) | per stage: total %.0f, wait full %.0f, mma issue %.0f, commit %.0f cyc\n", N, reuse, S, tma, ms,
                 flops / ms / 1e9, bytes / ms / 1e6, bytes / (ms * 1e-3) / nsm / 1.9e9, pr[0] / nst, pr[1] / nst, pr[2] / nst, pr[3] / nst);
        }
  return 0;
}
