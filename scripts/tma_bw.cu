// TMA / bulk-copy streaming throughput per SM (microbenchmark for the chain-kernel
// diagnosis): every CTA (one per SM) streams 16 KB stages
// through an S-deep SMEM ring from an L2-resident buffer, one elected thread
// producing and consuming (no compute), and reports bytes per cycle per SM for
//   (a) 2D tensor boxes {64 bf16, 128 rows} of a [rows][64] tensor  (128-B rows, contiguous box)
//   (b) the same box shape from a [rows][104] tensor                 (128-B pieces of 208-B rows)
//   (c) cp.async.bulk 16 KB contiguous                               (one request per stage)
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o scripts/tma_bw scripts/tma_bw.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void __launch_bounds__(32, 1) stream_kernel(const __grid_constant__ CUtensorMap map, const char* src,
                                                      int mode, int stages, int iters, int rows_total,
                                                      unsigned long long* cycles) {
  extern __shared__ __align__(1024) uint8_t smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + stages * 16384);
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  if (threadIdx.x != 0) return;
  const long long t0 = clock64();
  uint32_t phase_bits = 0;
  const int row0 = (blockIdx.x * 128) % (rows_total - 128);
  auto issue = [&](int i) {
    const int s = i % stages;
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(16384));
    const int row = (row0 + (i % 64) * 128) % (rows_total - 128);
    if (mode == 2) {
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                       su32(smem + s * 16384)),
                   "l"(src + (size_t)row * 128), "r"(16384), "r"(su32(&full[s]))
                   : "memory");
    } else {
      asm volatile(
          "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
              su32(smem + s * 16384)),
          "l"(reinterpret_cast<uint64_t>(&map)), "r"(su32(&full[s])), "r"(0), "r"(row)
          : "memory");
    }
  };
  for (int i = 0; i < stages; ++i) issue(i);
  for (int i = 0; i < iters; ++i) {
    const int s = i % stages;
    const uint32_t par = (phase_bits >> s) & 1u;
    asm volatile(
        "{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(
            su32(&full[s])),
        "r"(par)
        : "memory");
    phase_bits ^= 1u << s;
    if (i + stages < iters) issue(i + stages);
  }
  cycles[blockIdx.x] = clock64() - t0;
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int rows = 16384;   // 16384 x 208 B = 3.4 MB: L2-resident
  char* buf;
  cudaMalloc(&buf, (size_t)rows * 208 * 2);
  cudaMemset(buf, 1, (size_t)rows * 208 * 2);
  unsigned long long* cyc;
  cudaMalloc(&cyc, sms * sizeof(unsigned long long));
  PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", reinterpret_cast<void**>(&encode), cudaEnableDefault, &q);
  cudaFuncSetAttribute(stream_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
  const char* names[3] = {"2D box {64,128}, 128-B rows (contiguous)", "2D box {64,128} of 208-B rows       ",
                          "cp.async.bulk 16 KB contiguous        "};
  for (int mode = 0; mode < 3; ++mode) {
    CUtensorMap map;
    const cuuint64_t inner = mode == 1 ? 104 : 64;
    cuuint64_t dims[2] = {inner, (cuuint64_t)rows};
    cuuint64_t strides[1] = {inner * 2};
    cuuint32_t box[2] = {64, 128};
    cuuint32_t es[2] = {1, 1};
    encode(&map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
           CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    for (int nsm : {sms, sms / 2, sms / 4, 16})
    for (int stages : {4, 8}) {
      const int iters = 4000;
      stream_kernel<<<nsm, 32, stages * 16384 + 1024>>>(map, buf, mode, stages, 100, rows, cyc);
      stream_kernel<<<nsm, 32, stages * 16384 + 1024>>>(map, buf, mode, stages, iters, rows, cyc);
      cudaDeviceSynchronize();
      unsigned long long h[256];
      cudaMemcpy(h, cyc, nsm * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
      double avg = 0;
      for (int i = 0; i < nsm; ++i) avg += (double)h[i] / nsm;
      const double bpc = 16384.0 * iters / avg;
      printf("%s SMs %3d stages %2d: %6.1f B/cycle/SM  (%5.0f cycles per 16 KB stage, ~%.1f TB/s aggregate at 1.965 GHz)\n",
             names[mode], nsm, stages, bpc, avg / iters, bpc * nsm * 1.965e9 / 1e12);
    }
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
