// Microbenchmark: tcgen05.mma issue rate (cta_group::1 and ::2) on B200 (sm_100a).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mma2_issue scripts/mma2_issue.cu && ./mma2_issue
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(c));
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t par) {
  asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(
                   smem_u32(b)), "r"(par) : "memory");
}
__device__ int g_aw = 64;   // K atom width: 64 (SW128), 32 (SW64), 16 (SW32)
__device__ __forceinline__ uint64_t desc(uint32_t saddr) {   // K-major, swizzle per g_aw
  const int aw = 32;
  const uint64_t layout = aw == 64 ? 2 : aw == 32 ? 4 : 6;
  return (uint64_t)((saddr & 0x3FFFF) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(16 * aw >> 4) << 32) |
         ((uint64_t)1 << 46) | (layout << 61);
}
template <int CG>
__device__ __forceinline__ void mma(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  if (CG == 1)
    asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
                 "l"(a), "l"(b), "r"(idesc), "r"(acc));
  else
    asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
                 "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
template <int CG>
__device__ __forceinline__ void commit_nomc(uint64_t* b) {
  if (CG == 1)
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(b)) : "memory");
  else
    asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(b)) : "memory");
}
template <int CG>
__device__ __forceinline__ void commit(uint64_t* b) {
  if (CG == 1)
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(b)) : "memory");
  else
    asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(smem_u32(b)), "h"((uint16_t)3) : "memory");
}

__device__ int g_cev = 0, g_cmode = 0;
template <int CG>
__global__ void __cluster_dims__(CG, 1, 1) k(int iters, int N, int nw, int rot, unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* base = (uint8_t*)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar[4];
  __shared__ uint32_t slot;
  uint32_t rank = 0;
  if (CG == 2) asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  if (threadIdx.x < 32) {
    if (CG == 1) {
      asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&slot)));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    } else {
      asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&slot)));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    }
  }
  if (threadIdx.x == 0) {
    for (int i = 0; i < 4; ++i) mbar_init(&bar[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  for (int i = threadIdx.x; i < 4 * 49152 / 4; i += blockDim.x) ((uint32_t*)base)[i] = 0;
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t M = CG == 2 ? 256 : 128;
  const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
  const int w = threadIdx.x >> 5;
  const int cev = g_cev, awl = g_aw, cmode = g_cmode;
  if (rank == 0 && w < nw && (threadIdx.x & 31) == 0) {
    const uint32_t d = slot + (uint32_t)(w * (512 / nw));
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      // rot = 0: one A / B pair; rot > 0: A / B atoms rotate over `rot` distinct 24 KB stages
      const int st = rot ? (i % rot) : 0;
      const uint64_t a = desc(smem_u32(base + st * 49152)), b = desc(smem_u32(base + st * 49152 + 16384));
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        mma<CG>(d, a + 2 * (j & (awl / 16 - 1)), b + 2 * (j & (awl / 16 - 1)), idesc, (i | j) > 0);
        if (cev && (j % cev) == cev - 1) {
          if (cmode == 0) commit<CG>(&bar[2 + (j & 1)]);
          else commit_nomc<CG>(&bar[2 + (j & 1)]);
        }
      }
    }
    commit<CG>(&bar[w]);
    mbar_wait(&bar[w], 0);
    out[w] = clock64() - t0;
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (threadIdx.x < 32) {
    if (CG == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(slot));
    else asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(slot));
  }
}

int main() {
  unsigned long long* d;
  cudaMalloc(&d, 148 * 64);
  const int smem = 4 * 49152 + 2048;
  cudaFuncSetAttribute(k<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(k<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  for (int cmode : {0, 1})
  for (int cev : {0, 1, 8})
    for (int cg : {1, 2})
      for (int N : {128}) {
        cudaMemcpyToSymbol(g_cmode, &cmode, sizeof(int));
        int aw = 32;
        cudaMemcpyToSymbol(g_aw, &aw, sizeof(int));
        cudaMemcpyToSymbol(g_cev, &cev, sizeof(int));
        const int iters = 500, nw = 1, grid = 148, rot = 4;
        for (int rep = 0; rep < 2; ++rep) {
          if (cg == 1) k<1><<<grid, 128, smem>>>(iters, N, nw, rot, d);
          else k<2><<<grid, 128, smem>>>(iters, N, nw, rot, d);
        }
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
        unsigned long long c = 0;
        cudaMemcpy(&c, d, 8, cudaMemcpyDeviceToHost);
        const double per = (double)c / (iters * 8.0);
        const double floor_ = (cg == 2 ? 256.0 : 128.0) * N / (256.0 * cg);
        printf("multicast %d commit every %d MMAs, cta_group::%d N=%3d: %6.1f cyc per MMA, floor %5.1f -> %.2f\n", 1 - cmode, cev, cg, N, per, floor_, floor_ / per);
      }
  return 0;
}
