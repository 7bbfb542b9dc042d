// Microbenchmark: cost of tcgen05.commit inside a stream of cta_group::2 MMAs, issued the
// way kernels_pair.cu issues them (whole warp, elect.sync, tc_ptx.cuh wrappers).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_icpp_songljkj0024_b200/csrc -o scripts/commit_cost scripts/commit_cost.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>
#include "tc_ptx.cuh"
using namespace temco::ptx;

template <int CEV, int N>
__global__ void __cluster_dims__(2, 1, 1) k(int iters, unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* base = (uint8_t*)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar[4];
  __shared__ uint32_t slot;
  const uint32_t rank = cluster_ctarank();
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    for (int i = 0; i < 4; ++i) mbar_init(&bar[i], 1);
    fence_mbar_init_cluster();
  }
  for (int i = threadIdx.x; i < 4 * 32768 / 4; i += blockDim.x) ((uint32_t*)base)[i] = 0;
  asm volatile("fence.proxy.async.shared::cta;");
  tc_fence_before();
  cluster_sync_all();
  tc_fence_after();
  const uint32_t idesc = idesc_bf16(256, N);
  if (rank == 0 && threadIdx.x < 32) {
    const uint32_t d = slot;
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      const int st = i & 3;
      const uint64_t a = umma_desc_k(smem_u32(base + st * 32768), 32), b = umma_desc_k(smem_u32(base + st * 32768 + 16384), 32);
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        mma2_bf16_w(d + (uint32_t)((j >> 2) * 128), a + 2 * (j & 1), b + 2 * (j & 1), idesc, (i | (j & 3)) > 0);
        if (CEV && (j % (CEV ? CEV : 1)) == (CEV ? CEV : 1) - 1) mma2_commit_mc_w(&bar[2 + ((j / (CEV ? CEV : 1)) & 1)], 3);
      }
    }
    mma2_commit_mc_w(&bar[0], 3);
    mbar_wait(&bar[0], 0);
    if (threadIdx.x == 0) out[0] = clock64() - t0;
  }
  tc_fence_before();
  cluster_sync_all();
  if (threadIdx.x < 32) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(slot));
  }
}

template <int CEV, int N>
void run(unsigned long long* d) {
  const int smem = 4 * 32768 + 2048, iters = 500;
  cudaFuncSetAttribute(k<CEV, N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  for (int rep = 0; rep < 2; ++rep) k<CEV, N><<<148, 128, smem>>>(iters, d);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); exit(1); }
  unsigned long long c = 0;
  cudaMemcpy(&c, d, 8, cudaMemcpyDeviceToHost);
  printf("N=%3d commit every %d MMAs: %6.1f cycles per MMA (floor %d)\n", N, CEV, (double)c / (iters * 8.0), N / 2);
}

int main() {
  unsigned long long* d;
  cudaMalloc(&d, 64);
  run<0, 128>(d); run<8, 128>(d); run<4, 128>(d); run<2, 128>(d); run<1, 128>(d);
  run<0, 256>(d); run<8, 256>(d); run<4, 256>(d); run<1, 256>(d);
  run<0, 32>(d); run<8, 32>(d); run<1, 32>(d);
  return 0;
}
