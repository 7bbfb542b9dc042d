// tcgen05 GEMM + bias / ReLU epilogue (sm_100a); see gemm.h.
//
// CTA tile: 128 rows (M: images or pixels) x 256 outputs (N), fp32 accumulator in
// TMEM (256 columns).  Warp 0 lane 0 streams x [128 x 64] and W [256 x 64] atoms
// (TMA, SW128) through a 4-stage ring; warp 1 issues tcgen05.mma (M=128, N=256,
// K=16: 128 tensor cycles per instruction, 4 per stage); after the K loop all four
// warps drain TMEM (one row per thread, 32 columns per tcgen05.ld) and apply the
// epilogue.  splits > 1: each CTA of the z dimension owns a contiguous K range and
// writes fp32 partials; gemm_reduce_kernel sums them in split order (deterministic)
// and applies bias / ReLU.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstring>

#include "tmap.h"
#include "gemm.h"
#include "tc_ptx.cuh"

namespace temco {

namespace {
constexpr int kBM = 128, kBN = 256, kBK = 64;
constexpr int kStageA = kBM * kBK * 2, kStageB = kBN * kBK * 2, kStage = kStageA + kStageB;
constexpr int kGemmStages = 4;
constexpr int kGemmThreads = 128;

uint16_t to_bf16(float f) {
  uint32_t u;
  memcpy(&u, &f, 4);
  u += 0x7FFF + ((u >> 16) & 1);
  return (uint16_t)(u >> 16);
}
}  // namespace

bool gemm_lower(GemmDesc& d, const float* w, const std::vector<float>* bias, std::vector<uint16_t>& tcw,
                std::vector<float>& params, int64_t& ws_elems) {
  if (d.K % 8 || d.K <= 0 || d.O <= 0 || d.M <= 0) return false;
  if (d.x.where != W_ARENA || d.x.dtype != DT_BF16) return false;
  d.Opad = (d.O + kBN - 1) / kBN * kBN;
  while (tcw.size() % 512) tcw.push_back(0);
  d.w = (int64_t)tcw.size();
  tcw.resize(tcw.size() + (size_t)d.Opad * d.K, 0);
  for (int o = 0; o < d.O; ++o)
    for (int k = 0; k < d.K; ++k) tcw[d.w + (size_t)o * d.K + k] = to_bf16(w[(size_t)o * d.K + k]);
  d.b = -1;
  if (bias) {
    while (params.size() % 4) params.push_back(0.f);
    d.b = (int64_t)params.size();
    params.insert(params.end(), bias->begin(), bias->end());
  }
  // split K when the output tiles alone leave most SMs idle (weight-bound heads)
  const int katoms = (d.K + kBK - 1) / kBK;
  const int tiles = (d.Opad / kBN) * ((d.M + kBM - 1) / kBM);
  int splits = 1;
  while (tiles * splits * 2 <= 148 && katoms / (splits * 2) >= 8) splits *= 2;
  d.kper = (katoms + splits - 1) / splits;
  d.splits = (katoms + d.kper - 1) / d.kper;
  if (d.splits > 1) ws_elems = std::max<int64_t>(ws_elems, (int64_t)d.splits * d.M * d.Opad);
  d.stages = std::max(2, std::min(kGemmStages, d.kper));   // short K: smaller ring, 2 CTAs per SM
  d.smem_bytes = 1024 + d.stages * kStage + 256;
  d.alg_flops = 2LL * d.M * d.K * d.O;
  d.alg_bytes = 2LL * d.M * d.K + 2LL * d.O * d.K + (int64_t)d.M * d.O * (d.y.dtype == DT_F32 ? 4 : 2);
  return true;
}

bool gemm_finalize(GemmDesc& d, char* arena, uint16_t* tcw, std::string& err) {
  const auto encode = tmap_encoder(err);
  if (!encode) return false;
  auto make = [&](unsigned char* dst, void* base, uint64_t inner, uint64_t outer, uint32_t box_outer) {
    cuuint64_t dims[2] = {inner, outer};
    cuuint64_t strides[1] = {inner * 2};
    cuuint32_t box[2] = {(cuuint32_t)kBK, box_outer};
    cuuint32_t es[2] = {1, 1};
    return encode(reinterpret_cast<CUtensorMap*>(dst), CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, base, dims, strides, box,
                  es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
  };
  if (!make(d.amap, arena + d.x.off, (uint64_t)d.K, (uint64_t)d.M, kBM) ||
      !make(d.bmap, tcw + d.w, (uint64_t)d.K, (uint64_t)d.Opad, kBN)) {
    err = "cuTensorMapEncodeTiled failed (gemm)";
    return false;
  }
  return true;
}

namespace {
using namespace ptx;

// output element index of GEMM entry (m, o): row-major [M x O], or the pixel-shuffle
// position of a stride-k transposed conv
__device__ __forceinline__ int64_t out_index(const GemmDesc& d, int64_t m, int o) {
  if (!d.shuffle_k) return m * d.O + o;
  const int k = d.shuffle_k;
  const int tap = o / d.sh_Co, oc = o - tap * d.sh_Co, i = tap / k, j = tap - i * k;
  const int64_t w = m % d.sh_W, t = m / d.sh_W, h = t % d.sh_H, n = t / d.sh_H;
  return (((n * d.sh_H * k + h * k + i) * (int64_t)d.sh_W * k) + w * k + j) * d.sh_Co + oc;
}

__device__ __forceinline__ void store_out(void* y, int dtype, int64_t i, float v) {
  if (dtype == DT_F32)
    static_cast<float*>(y)[i] = v;
  else
    static_cast<__nv_bfloat16*>(y)[i] = __float2bfloat16_rn(v);
}

__global__ void __launch_bounds__(kGemmThreads, 1) gemm_kernel(const __grid_constant__ GemmDesc d, RunPtrs p, float* ws) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  const int S = d.stages;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + S * kStage);
  uint64_t* empty = full + S;
  uint64_t* done = empty + S;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(done + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n0 = blockIdx.x * kBN, m0 = blockIdx.y * kBM;
  const int katoms = (d.K + kBK - 1) / kBK;
  const int a0 = blockIdx.z * d.kper, a1 = min(katoms, a0 + d.kper);
  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    mbar_init(done, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(smem_u32(tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tslot;
  pdl_wait();
  if (warp == 0) {
    if (lane == 0) {   // TMA producer
      int st = 0;
      uint32_t ph = 0;
      for (int a = a0; a < a1; ++a) {
        mbar_wait(&empty[st], ph ^ 1);
        mbar_expect_tx(&full[st], kStage);
        uint8_t* s = smem + st * kStage;
        tma_load_2d(s, d.amap, &full[st], a * kBK, m0);
        tma_load_2d(s + kStageA, d.bmap, &full[st], a * kBK, n0);
        if (++st == S) st = 0, ph ^= 1;
      }
    }
  } else if (warp == 1) {   // MMA issuer
    const uint32_t idesc = idesc_bf16(kBM, kBN);
    int st = 0;
    uint32_t ph = 0;
    for (int a = a0; a < a1; ++a) {
      mbar_wait(&full[st], ph);
      tc_fence_after();
      const uint32_t sa = smem_u32(smem + st * kStage);
      const uint64_t ad = umma_desc(sa), bd = umma_desc(sa + kStageA);
      for (int k = 0; k < kBK / 16; ++k) mma_bf16_w(tbase, ad + 2 * k, bd + 2 * k, idesc, (a > a0 || k > 0) ? 1u : 0u);
      mma_commit_w(&empty[st]);
      if (++st == S) st = 0, ph ^= 1;
    }
    mma_commit_w(done);
  }
  // epilogue: all four warps, one accumulator row (TMEM lane) per thread
  mbar_wait(done, 0);
  tc_fence_after();
  const int row = warp * 32 + lane, m = m0 + row;
  const uint32_t trow = tbase + ((uint32_t)(warp * 32) << 16);
  void* y = const_cast<void*>(loc_ptr(d.y, p));
  void* y2 = d.y2.where >= 0 ? const_cast<void*>(loc_ptr(d.y2, p)) : nullptr;
  const bool vec8 = d.y.dtype == DT_BF16 && (y2 == nullptr || d.y2.dtype == DT_BF16) &&
                    (d.shuffle_k ? d.sh_Co % 8 == 0 : d.O % 8 == 0);
  for (int c = 0; c < kBN; c += 32) {
    uint32_t v[32];
    tmem_ld32(trow + c, v);
    tmem_wait_ld();
    if (m >= d.M) continue;
    if (d.splits > 1) {   // fp32 partial of this K range: ws[split][m][o], o < Opad
      float4* dst = reinterpret_cast<float4*>(ws + ((int64_t)blockIdx.z * d.M + m) * d.Opad + n0 + c);
#pragma unroll
      for (int i = 0; i < 8; ++i)
        dst[i] = make_float4(__uint_as_float(v[4 * i]), __uint_as_float(v[4 * i + 1]), __uint_as_float(v[4 * i + 2]),
                             __uint_as_float(v[4 * i + 3]));
      continue;
    }
    if (vec8) {   // bf16 output, 8 consecutive channels per 16-byte store
#pragma unroll
      for (int g8 = 0; g8 < 4; ++g8) {
        const int o = n0 + c + g8 * 8;
        if (o >= d.O) break;
        float f[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          f[i] = __uint_as_float(v[g8 * 8 + i]) + (d.b >= 0 ? p.params[d.b + o + i] : 0.f);
          if (d.relu) f[i] = fmaxf(f[i], 0.f);
        }
        const int64_t oi = out_index(d, m, o);
        *reinterpret_cast<uint4*>(static_cast<__nv_bfloat16*>(y) + oi) =
            make_uint4(pack_bf16(f[0], f[1]), pack_bf16(f[2], f[3]), pack_bf16(f[4], f[5]), pack_bf16(f[6], f[7]));
        if (y2)
          *reinterpret_cast<uint4*>(static_cast<__nv_bfloat16*>(y2) + oi) =
              make_uint4(pack_bf16(fmaxf(f[0], 0.f), fmaxf(f[1], 0.f)), pack_bf16(fmaxf(f[2], 0.f), fmaxf(f[3], 0.f)),
                         pack_bf16(fmaxf(f[4], 0.f), fmaxf(f[5], 0.f)), pack_bf16(fmaxf(f[6], 0.f), fmaxf(f[7], 0.f)));
      }
      continue;
    }
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      const int o = n0 + c + i;
      if (o >= d.O) break;
      float x = __uint_as_float(v[i]) + (d.b >= 0 ? p.params[d.b + o] : 0.f);
      if (d.relu) x = fmaxf(x, 0.f);
      store_out(y, d.y.dtype, out_index(d, m, o), x);
      if (y2) store_out(y2, d.y2.dtype, out_index(d, m, o), fmaxf(x, 0.f));
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tbase));
  }
}

// y[m, o] = act(sum_s ws[s][m][o] + b[o]) -- partial sums in split order (deterministic)
__global__ void gemm_reduce_kernel(const __grid_constant__ GemmDesc d, RunPtrs p, const float* ws) {
  pdl_wait();
  void* y = const_cast<void*>(loc_ptr(d.y, p));
  void* y2 = d.y2.where >= 0 ? const_cast<void*>(loc_ptr(d.y2, p)) : nullptr;
  const int64_t total = (int64_t)d.M * d.O;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t m = i / d.O;
    const int o = (int)(i - m * d.O);
    float x = d.b >= 0 ? p.params[d.b + o] : 0.f;
    for (int s = 0; s < d.splits; ++s) x += ws[((int64_t)s * d.M + m) * d.Opad + o];
    if (d.relu) x = fmaxf(x, 0.f);
    store_out(y, d.y.dtype, out_index(d, m, o), x);
    if (y2) store_out(y2, d.y2.dtype, out_index(d, m, o), fmaxf(x, 0.f));
  }
}

}  // namespace

void launch_gemm(const GemmDesc& d, const RunPtrs& p, float* ws, cudaStream_t s) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(gemm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    attr = true;
  }
  launch_pdl(gemm_kernel, dim3(d.Opad / kBN, (d.M + kBM - 1) / kBM, d.splits), dim3(kGemmThreads), d.smem_bytes, s, d,
             p, ws);
  if (d.splits > 1) {
    const int64_t total = (int64_t)d.M * d.O;
    const int grid = (int)std::min<int64_t>((total + 255) / 256, 148LL * 8);
    launch_pdl(gemm_reduce_kernel, dim3(grid), dim3(256), 0, s, d, p, (const float*)ws);
  }
}

}  // namespace temco
