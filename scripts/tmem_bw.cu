// Microbenchmark: tcgen05.ld / tcgen05.st throughput per SM on B200 (sm_100a).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tmem_bw scripts/tmem_bw.cu && ./tmem_bw
// One CTA per SM, W warps; warp w reads TMEM lane quarter w % 4, columns
// ((w / 4) * 32 + i * 32 * (W/4)) mod 512, 32 columns (4 KB) per instruction.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

#define R32(v) "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), \
  "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),          \
  "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),         \
  "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
#define I32(v) "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), \
  "r"(v[8]), "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15]),          \
  "r"(v[16]), "r"(v[17]), "r"(v[18]), "r"(v[19]), "r"(v[20]), "r"(v[21]), "r"(v[22]), "r"(v[23]),         \
  "r"(v[24]), "r"(v[25]), "r"(v[26]), "r"(v[27]), "r"(v[28]), "r"(v[29]), "r"(v[30]), "r"(v[31])

template <int MODE>  // 0 ld, 1 st, 2 ld+st (read-modify-write, ReLU)
__global__ void k(int iters, int depth, unsigned long long* cyc, float* sink) {
  __shared__ uint32_t slot;
  const int warp = threadIdx.x / 32, nw = blockDim.x / 32;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t base = slot + ((uint32_t)((warp & 3) * 32) << 16);
  const int groups = nw / 4;
  const int g = warp / 4;
  uint32_t v[32];
  for (int i = 0; i < 32; ++i) v[i] = threadIdx.x + i;
  float acc = 0.f;
  __syncthreads();
  const unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    for (int d = 0; d < depth; ++d) {
      const uint32_t col = (uint32_t)(((g + (it * depth + d) * groups) * 32) & 511);
      if (MODE == 0 || MODE == 2) {
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                     "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                     : R32(v) : "r"(base + col));
      }
      if (MODE == 2) {
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
        for (int i = 0; i < 32; ++i) v[i] = __float_as_uint(fmaxf(__uint_as_float(v[i]), 0.f));
      }
      if (MODE == 1 || MODE == 2) {
        asm volatile("tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,"
                     "%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};"
                     ::"r"(base + col), I32(v) : "memory");
      }
    }
    if (MODE == 0) {
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
      for (int i = 0; i < 32; ++i) acc += __uint_as_float(v[i]);
    } else {
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    }
  }
  const unsigned long long t1 = clock64();
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
  sink[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(slot));
}

int main() {
  unsigned long long* cyc;
  float* sink;
  cudaMalloc(&cyc, 148 * 8);
  cudaMalloc(&sink, 148 * 1024 * 4);
  unsigned long long h[148];
  const char* names[3] = {"ld", "st", "ld+relu+st"};
  for (int mode = 0; mode < 3; ++mode)
    for (int nw : {4, 8, 16})
      for (int depth : {1, 2, 4}) {
        const int iters = 2000;
        for (int rep = 0; rep < 2; ++rep) {
          if (mode == 0) k<0><<<148, nw * 32>>>(iters, depth, cyc, sink);
          if (mode == 1) k<1><<<148, nw * 32>>>(iters, depth, cyc, sink);
          if (mode == 2) k<2><<<148, nw * 32>>>(iters, depth, cyc, sink);
        }
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
        cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
        double c = 0;
        for (int i = 0; i < 148; ++i) c += h[i];
        c /= 148;
        const double bytes = (double)iters * depth * nw * 32 * 32 * 4;   // per SM, per direction
        printf("%-11s warps %2d depth %d: %8.0f cyc, %6.1f B/cyc/SM\n", names[mode], nw, depth, c, bytes / c);
      }
  return 0;
}
