// Microbenchmark: what slows a single tcgen05 issuer warp inside a warp-specialised kernel?
// Blocks of 4 cta_group::2 MMAs (N=128, one asm block each, like kernels_pair.cu), with
//   WAIT: an mbarrier try_wait on an already-completed phase before every block;
//   BUSY: 16 other warps of the CTA either spin on try_wait of a never-completing phase (1),
//         or run dependent FP math (2);
//   COMMIT: a multicast commit after every block.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_icpp_songljkj0024_b200/csrc -o scripts/issue_cost scripts/issue_cost.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>
#include "tc_ptx.cuh"
using namespace temco::ptx;

__device__ float g_sink;

template <int WAIT, int BUSY, int COMMIT>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(18 * 32, 1) k(int iters, unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* base = (uint8_t*)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar[6];
  __shared__ uint32_t slot;
  __shared__ volatile int stop;
  const uint32_t rank = cluster_ctarank();
  const int warp = threadIdx.x >> 5;
  if (warp == 17) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    for (int i = 0; i < 6; ++i) mbar_init(&bar[i], 1);
    stop = 0;
    fence_mbar_init_cluster();
  }
  for (int i = threadIdx.x; i < 4 * 32768 / 4; i += blockDim.x) ((uint32_t*)base)[i] = 0;
  asm volatile("fence.proxy.async.shared::cta;");
  tc_fence_before();
  cluster_sync_all();
  tc_fence_after();
  if (threadIdx.x == 0) mbar_arrive(&bar[4]);   // bar[4]: phase 0 completed (WAIT target)
  __syncthreads();
  const uint32_t idesc = idesc_bf16(256, 128);
  if (warp == 17) {
    if (rank == 0) {
      const uint32_t hi = udesc_hi(32);
      long long t0 = clock64();
      for (int i = 0; i < iters; ++i) {
        const int st = i & 3;
        const uint32_t a = udesc_lo(smem_u32(base + st * 32768)), b = udesc_lo(smem_u32(base + st * 32768 + 16384));
        if (WAIT) {
          mbar_wait_u(&bar[4], 0);
          tc_fence_after();
        }
        mma2_k4_w(slot + (uint32_t)((i & 1) * 128), a, hi, b, hi, idesc, i > 1, 2);
        if (COMMIT) mma2_commit_mc_w(&bar[2 + (i & 1)], 3);
      }
      mma2_commit_mc_w(&bar[0], 3);
      mbar_wait(&bar[0], 0);
      if (threadIdx.x == 32 * 17) out[0] = clock64() - t0;
    }
    if (threadIdx.x == 32 * 17) stop = 1;
  } else if (warp < 16) {
    if (BUSY == 1) {
      while (!stop) mbar_try_wait(&bar[5], 0);
    } else if (BUSY == 2) {
      float x = threadIdx.x;
      while (!stop)
        for (int j = 0; j < 64; ++j) x = fmaf(x, 1.0001f, 0.5f);
      if (x == 1.2345f) g_sink = x;
    }
  }
  __syncthreads();
  tc_fence_before();
  cluster_sync_all();
  if (warp == 17) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(slot));
  }
}

template <int WAIT, int BUSY, int COMMIT>
void run(unsigned long long* d) {
  const int smem = 4 * 32768 + 2048, iters = 2000;
  cudaFuncSetAttribute(k<WAIT, BUSY, COMMIT>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  for (int rep = 0; rep < 2; ++rep) k<WAIT, BUSY, COMMIT><<<148, 18 * 32, smem>>>(iters, d);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); exit(1); }
  unsigned long long c = 0;
  cudaMemcpy(&c, d, 8, cudaMemcpyDeviceToHost);
  printf("wait=%d busy=%d commit=%d: %7.1f cycles per 2-MMA block (tensor floor 128)\n", WAIT, BUSY, COMMIT, (double)c / iters);
}

int main() {
  unsigned long long* d;
  cudaMalloc(&d, 64);
  run<0, 0, 0>(d); run<0, 0, 1>(d); run<1, 0, 0>(d); run<1, 0, 1>(d);
  run<0, 1, 0>(d); run<1, 1, 1>(d); run<0, 2, 0>(d); run<1, 2, 1>(d);
  return 0;
}
