// Microbenchmark: tcgen05.ld latency / bandwidth for 16 epilogue warps while a single
// thread keeps the tensor core busy with MMAs into other TMEM columns (B200, sm_100a).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tmem_contention scripts/tmem_contention.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t saddr) {
  return (uint64_t)((saddr & 0x3FFFF) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) | ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__device__ __forceinline__ void mma(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d), "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
#define R32(v) "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])

__global__ void __launch_bounds__(544, 1) k(int iters, int mma_on, int N, int depth, unsigned long long* out, float* sink) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* base = (uint8_t*)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
  __shared__ uint32_t slot;
  __shared__ volatile int stop;
  __shared__ int ndone;
  const int w = threadIdx.x >> 5;
  if (w == 16) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) stop = 0, ndone = 0;
  for (int i = threadIdx.x; i < 65536 / 4; i += blockDim.x) ((uint32_t*)base)[i] = 0;
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tb = slot;
  if (w == 16) {
    if (mma_on && (threadIdx.x & 31) == 0) {
      const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
      const uint64_t a = desc(smem_u32(base)), b = desc(smem_u32(base + 32768));
      int i = 0;
      while (!stop) {   // accumulate into columns [0, 384) (buffers 0-2); the epilogue reads [384, 512)
        for (int j = 0; j < 8; ++j) mma(tb + (uint32_t)(((i + j) % 3) * 128), a + 2 * (j & 3), b + 2 * (j & 3), idesc, 1);
        ++i;
      }
    }
  } else {
    const int q = w & 3, g = w >> 2;
    const uint32_t ta = tb + ((uint32_t)(q * 32) << 16) + 384 + g * 32;
    float acc = 0.f;
    uint32_t v[32];
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
      for (int dd = 0; dd < depth; ++dd)
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                     : R32(v) : "r"(ta));
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
      for (int i = 0; i < 32; ++i) acc += __uint_as_float(v[i]);
    }
    long long t1 = clock64();
    if ((threadIdx.x & 31) == 0) {
      out[blockIdx.x * 16 + w] = t1 - t0;
      if (atomicAdd(&ndone, 1) == 15) stop = 1;
    }
    sink[threadIdx.x] = acc;
  }
  __syncthreads();
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (w == 16) {
    asm volatile("tcgen05.fence::after_thread_sync;");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tb));
  }
}

int main() {
  unsigned long long* d;
  float* sink;
  cudaMalloc(&d, 148 * 16 * 8);
  cudaMalloc(&sink, 4096 * 4);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 70000);
  for (int mma_on : {0, 1})
    for (int N : {128, 256})
      for (int depth : {1, 2}) {
        if (!mma_on && N == 256) continue;
        const int iters = 2000;
        k<<<148, 544, 70000>>>(iters, mma_on, N, depth, d, sink);
        k<<<148, 544, 70000>>>(iters, mma_on, N, depth, d, sink);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
        unsigned long long h[148 * 16];
        cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
        double mx = 0;
        for (int i = 0; i < 148 * 16; ++i) mx = h[i] > mx ? h[i] : mx;
        const double per = mx / iters;
        printf("mma_on=%d N=%3d depth=%d: %7.1f cycles per round (16 warps x %d x 4 KB) = %6.1f B/cycle/SM\n", mma_on, N, depth,
               per, depth, 16.0 * depth * 4096 / per);
      }
  return 0;
}
