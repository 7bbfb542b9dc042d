// Microbenchmark: cost of tcgen05.commit -> mbarrier handoffs on B200 (sm_100a).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o commit_bench scripts/commit_bench.cu && ./commit_bench
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(c));
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t par) {
  asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(
                   smem_u32(b)),
               "r"(par)
               : "memory");
}
__device__ __forceinline__ void commit(uint64_t* b) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(b))
               : "memory");
}
__device__ __forceinline__ void mma(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
               "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ uint64_t desc(uint32_t saddr) {   // K-major SW128
  return (uint64_t)((saddr & 0x3FFFF) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}

__global__ void k(int mode, int iters, int nmma, int N, unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* base = (uint8_t*)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar[2];
  __shared__ uint32_t slot;
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], mode == 1 ? iters : 1);
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  for (int i = threadIdx.x; i < 65536 / 4; i += blockDim.x) ((uint32_t*)base)[i] = 0;
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
  if (threadIdx.x == 0) {
    const uint64_t a = desc(smem_u32(base)), b = desc(smem_u32(base + 32768));
    long long t0 = clock64();
    if (mode == 0) {          // round trip: [nmma MMAs] commit, wait
      for (int i = 0; i < iters; ++i) {
        for (int j = 0; j < nmma; ++j) mma(slot, a + 2 * (j & 3), b + 2 * (j & 3), idesc, j > 0);
        commit(&bar[0]);
        mbar_wait(&bar[0], i & 1);
      }
    } else if (mode == 1) {   // issue rate of commits (one barrier phase at the end)
      for (int i = 0; i < iters; ++i) {
        for (int j = 0; j < nmma; ++j) mma(slot, a + 2 * (j & 3), b + 2 * (j & 3), idesc, j > 0);
        commit(&bar[1]);
      }
      mbar_wait(&bar[1], 0);
    } else {                  // MMA issue rate, one commit at the end
      for (int i = 0; i < iters; ++i)
        for (int j = 0; j < nmma; ++j) mma(slot, a + 2 * (j & 3), b + 2 * (j & 3), idesc, j > 0);
      commit(&bar[0]);
      mbar_wait(&bar[0], 0);
    }
    out[0] = clock64() - t0;
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(slot));
}

int main() {
  unsigned long long* d;
  cudaMalloc(&d, 8);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 70000);
  const char* names[3] = {"roundtrip (mma* commit wait)", "commit issue (mma* commit)", "mma issue only"};
  for (int mode = 0; mode < 3; ++mode)
    for (int N : {64, 128, 256})
      for (int nmma : {0, 1, 2, 4, 8}) {
        if (mode == 2 && nmma == 0) continue;
        const int iters = 1000;
        k<<<1, 128, 70000>>>(mode, iters, nmma, N, d);
        k<<<1, 128, 70000>>>(mode, iters, nmma, N, d);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
        unsigned long long c;
        cudaMemcpy(&c, d, 8, cudaMemcpyDeviceToHost);
        printf("%-30s N=%3d nmma=%d: %8.1f cyc/iter  (%6.1f cyc/mma; floor %d)\n", names[mode], N, nmma,
               (double)c / iters, nmma ? (double)c / iters / nmma : 0.0, 128 * N / 256);
      }
  return 0;
}
