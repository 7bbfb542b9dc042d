// Per-SM L2 -> SMEM ingress: TMA bulk copies vs cp.async (LSU path) vs both at once
// (does the LSU path add bandwidth on top of the TMA cap measured by tma_bw.cu?).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o scripts/ingress_bw scripts/ingress_bw.cu
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// warp 0: TMA 1-D bulk copies of 16 KB through an 8-stage ring (if use_tma)
// warps 1..W: cp.async 16-B copies of 16 KB per iteration into their own buffer (if use_lsu)
__global__ void __launch_bounds__(32 * 9, 1) ingress_kernel(const char* src, int use_tma, int use_lsu, int iters,
                                                           unsigned long long* out, int windows) {
  extern __shared__ __align__(1024) uint8_t smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + 8 * 16384 + 16384);
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  if (threadIdx.x == 0) {
    for (int s = 0; s < 8; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const size_t span = 1u << 20;   // 1 MB windows; CTAs sharing a window read the same lines
  const char* base = src + (size_t)(blockIdx.x % windows) * span;
  const long long t0 = clock64();
  if (warp == 0 && use_tma && lane == 0) {
    uint32_t ph = 0;
    for (int i = 0; i < iters + 8; ++i) {
      const int s = i % 8;
      if (i >= 8) {
        asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(
                         su32(&full[s])), "r"((ph >> s) & 1u) : "memory");
        ph ^= 1u << s;
      }
      if (i < iters) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(16384));
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                         su32(smem + s * 16384)), "l"(base + (size_t)(i % 64) * 16384), "r"(16384), "r"(su32(&full[s]))
                     : "memory");
      }
    }
  } else if (warp >= 1 && use_lsu) {
    // 8 warps x 2 KB per iteration = 16 KB per iteration, 4 groups in flight
    uint8_t* dst = smem + 8 * 16384 + (warp - 1) * 2048;
    for (int i = 0; i < iters; ++i) {
      const char* sp = base + (size_t)(i % 64) * 16384 + (warp - 1) * 2048;
#pragma unroll
      for (int k = 0; k < 4; ++k)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su32(dst + k * 512 + lane * 16)),
                     "l"(sp + k * 512 + lane * 16) : "memory");
      asm volatile("cp.async.commit_group;" ::: "memory");
      asm volatile("cp.async.wait_group 3;" ::: "memory");
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = clock64() - t0;
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  char* buf;
  cudaMalloc(&buf, 160u << 20);
  cudaMemset(buf, 1, 160u << 20);
  unsigned long long* cyc;
  cudaMalloc(&cyc, sms * sizeof(unsigned long long));
  cudaFuncSetAttribute(ingress_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
  const int smem = 9 * 16384 + 1024;
  const int iters = 4000;
  const char* names[3] = {"TMA bulk only   ", "cp.async only   ", "TMA + cp.async  "};
  for (int windows : {1, 8, 148})
  for (int m = 0; m < 3; ++m) {
    const int t = m != 1, l = m != 0;
    ingress_kernel<<<sms, 32 * 9, smem>>>(buf, t, l, 100, cyc, windows);
    ingress_kernel<<<sms, 32 * 9, smem>>>(buf, t, l, iters, cyc, windows);
    cudaDeviceSynchronize();
    unsigned long long h[256];
    cudaMemcpy(h, cyc, sms * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < sms; ++i) avg += (double)h[i] / sms;
    const double bytes = 16384.0 * iters * (t + l);
    printf("windows %3d %s %6.1f B/cycle/SM (%.1f TB/s over %d SMs)\n", windows, names[m], bytes / avg,
           bytes / avg * sms * 1.965e9 / 1e12, sms);
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
