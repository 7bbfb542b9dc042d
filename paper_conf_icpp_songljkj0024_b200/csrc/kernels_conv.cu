// tcgen05 implicit-GEMM convolution (see conv_tc.h).
//
// Per 128-output-pixel tile: the im2col rows are gathered straight from the
// NHWC input into the SW128 K-major SMEM layout (4 gather warps, 16-byte
// cp.async with zero-fill for padding taps, completion signalled on an
// mbarrier), the whole weight matrix stays resident in SMEM (one TMA load per
// CTA), one thread issues tcgen05.mma (M=128, N=Np, K=16) into one of two TMEM
// accumulators, and 4 epilogue warps drain TMEM -> bias -> bf16 -> global while
// the next tile accumulates.  The small-rank convolutions are HBM-bound (AI ~
// 25-40 flop/B); the tensor cores only have to keep up with the gather.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cudaTypedefs.h>

#include <algorithm>

#include "tmap.h"
#include "conv_tc.h"
#include "tc_ptx.cuh"

namespace temco {

namespace {

uint16_t f2bf(float f) {
  uint32_t u;
  memcpy(&u, &f, 4);
  u += 0x7FFF + ((u >> 16) & 1);
  return (uint16_t)(u >> 16);
}

}  // namespace

bool conv_tc_lower(const IR& ir, int out, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                   std::vector<float>& params, ConvTcDesc& d) {
  const Node& v = ir.nodes[out];
  if (v.op != OP_CONV || v.groups != 1) return false;
  const Node& x = ir.nodes[ir.oin[out][0]];
  const Loc& xl = loc.at(x.id);
  const Loc& yl = loc.at(out);
  if (xl.dtype != DT_BF16 || yl.dtype != DT_BF16 || yl.where != W_ARENA) return false;
  if (v.C % 8) return false;
  d = ConvTcDesc();
  d.x = xl;
  d.y = yl;
  d.N = ir.batch; d.H = x.H; d.W = x.W; d.Cin = x.C;
  d.Ho = v.H; d.Wo = v.W; d.kh = v.kh; d.kw = v.kw; d.sh = v.sh; d.sw = v.sw; d.ph = v.ph; d.pw = v.pw;
  d.Nout = v.C;
  d.vec = x.C % 8 == 0 ? 1 : 0;
  d.K = v.kh * v.kw * x.C;
  d.kchunks = (d.K + 7) / 8;
  d.katoms = (d.K + 63) / 64;
  d.npix = (int64_t)ir.batch * v.H * v.W;
  d.ntiles = (int)((d.npix + 127) / 128);
  d.taps = v.kh * v.kw;
  d.s = v.sh;
  // TMA mode: 16-byte channel rows, square stride / padding, strided boxes <= 256
  d.tma = (x.C % 8 == 0 && v.sh == v.sw && v.ph == v.pw && xl.where == W_ARENA) ? 1 : 0;
  if (d.tma) {
    d.kpt = (x.C + 63) / 64;
    d.katoms = d.taps * d.kpt;
    d.tw = std::min(v.W, 128);
    d.th = std::min(v.H, 128 / d.tw);
    d.tn = (d.th == v.H && d.tw == v.W) ? std::max(1, std::min(ir.batch, 128 / (v.H * v.W))) : 1;
    d.nwb = (v.W + d.tw - 1) / d.tw;
    d.nhb = (v.H + d.th - 1) / d.th;
    d.nnb = (ir.batch + d.tn - 1) / d.tn;
    d.mused = d.tw * d.th * d.tn;
    d.ntiles = d.nnb * d.nhb * d.nwb;
    if (d.tw * d.s > 256 || d.th * d.s > 256) d.tma = 0;
  }
  if (!d.tma) d.katoms = (d.K + 63) / 64;
  // fewest output-channel slices whose resident weight block fits the SMEM budget
  for (d.nsl = (v.C + 255) / 256;; ++d.nsl) {
    d.Nsl = ((v.C + d.nsl - 1) / d.nsl + 7) / 8 * 8;
    d.Np = (d.Nsl + 15) / 16 * 16;
    if (d.katoms * d.Np * 128 <= 112 * 1024) break;
    if (d.Nsl <= 8 || d.nsl >= 16) return false;
  }
  d.nsl = (v.C + d.Nsl - 1) / d.Nsl;
  const int wbytes = d.katoms * d.Np * 128;
  const int Kp = d.katoms * 64;
  std::vector<uint16_t> w((size_t)d.nsl * d.Np * Kp, 0);
  const std::vector<float>& src = *v.w;   // OIHW
  for (int o = 0; o < v.C; ++o)
    for (int c = 0; c < x.C; ++c)
      for (int a = 0; a < v.kh; ++a)
        for (int b = 0; b < v.kw; ++b) {
          // TMA mode: k = (tap * kpt + c / 64) * 64 + c % 64; gather mode: k = tap * Cin + c
          const int tap = a * v.kw + b;
          const size_t k = d.tma ? (size_t)(tap * d.kpt) * 64 + c : (size_t)tap * x.C + c;
          const size_t row = (size_t)(o / d.Nsl) * d.Np + o % d.Nsl;
          w[row * Kp + k] = f2bf(src[(((size_t)o * x.C + c) * v.kh + a) * v.kw + b]);
        }
  while (tcw.size() % 512) tcw.push_back(0);
  d.w = (int64_t)tcw.size();
  tcw.insert(tcw.end(), w.begin(), w.end());
  d.b = -1;
  if (v.b) {
    while (params.size() % 4) params.push_back(0.f);
    d.b = (int64_t)params.size();
    params.insert(params.end(), v.b->begin(), v.b->end());
  }
  d.stages = std::min(8, (220 * 1024 - wbytes) / 16384);
  if (d.stages < 2) return false;
  d.smem_bytes = 1024 + wbytes + d.stages * 16384 + 256;
  const int cols = 2 * d.Np;
  d.tmem_cols = cols <= 32 ? 32 : cols <= 64 ? 64 : cols <= 128 ? 128 : cols <= 256 ? 256 : 512;
  d.alg_flops = 2 * d.npix * (int64_t)d.K * d.Nout;
  d.alg_bytes = 2 * ((int64_t)d.N * d.H * d.W * d.Cin + d.npix * d.Nout);
  return true;
}

bool conv_tc_finalize(ConvTcDesc& d, uint16_t* tcw, std::string& err) {
  const auto encode = tmap_encoder(err);
  if (!encode) return false;
  const uint64_t Kp = (uint64_t)d.katoms * 64;
  cuuint64_t dims[2] = {Kp, (cuuint64_t)d.nsl * d.Np};
  cuuint64_t strides[1] = {Kp * 2};
  cuuint32_t box[2] = {64, (cuuint32_t)d.Np};
  cuuint32_t es[2] = {1, 1};
  CUresult r = encode(reinterpret_cast<CUtensorMap*>(d.wmap), CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, tcw + d.w, dims,
                      strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    err = "cuTensorMapEncodeTiled failed (conv weights)";
    return false;
  }
  return true;
}

bool conv_tc_finalize_x(ConvTcDesc& d, const void* x, std::string& err) {
  if (!d.tma) return true;
  const auto encode = tmap_encoder(err);
  if (!encode) return false;
  cuuint64_t dims[4] = {(cuuint64_t)d.Cin, (cuuint64_t)d.W, (cuuint64_t)d.H, (cuuint64_t)d.N};
  cuuint64_t strides[3] = {(cuuint64_t)d.Cin * 2, (cuuint64_t)d.W * d.Cin * 2, (cuuint64_t)d.H * d.W * d.Cin * 2};
  cuuint32_t box[4] = {64, (cuuint32_t)(d.tw * d.s), (cuuint32_t)(d.th * d.s), (cuuint32_t)d.tn};
  cuuint32_t es[4] = {1, (cuuint32_t)d.s, (cuuint32_t)d.s, 1};
  CUresult r = encode(reinterpret_cast<CUtensorMap*>(d.xmap), CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(x),
                      dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    err = "cuTensorMapEncodeTiled failed (conv input)";
    return false;
  }
  return true;
}

namespace {

using namespace ptx;

constexpr int kGatherWarps = 8;
constexpr int kConvThreads = 32 * (5 + kGatherWarps);   // warps 0-3 epilogue, 4..11 gather, 12 MMA

__global__ void __launch_bounds__(kConvThreads, 1) conv_tc_kernel(const __grid_constant__ ConvTcDesc d, RunPtrs p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  const int S = d.stages;
  const int wbytes = d.katoms * d.Np * 128;
  uint8_t* wres = smem;
  uint8_t* ring = smem + wbytes;
  uint64_t* bars = reinterpret_cast<uint64_t*>(ring + S * 16384);
  uint64_t* full = bars;
  uint64_t* empty = bars + S;
  uint64_t* acc_full = bars + 2 * S;
  uint64_t* acc_empty = acc_full + 2;
  uint64_t* wbar = acc_empty + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(wbar + 1);
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 32);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&acc_full[b], 1);
      mbar_init(&acc_empty[b], 4);
    }
    mbar_init(wbar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(d.tmem_cols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tmem_slot;
  const int hw = d.Ho * d.Wo;

  if (warp >= 4 && warp < 4 + kGatherWarps) {
    // ------------------------------------------------------------ im2col gather
    // warp-per-stage: gather warp gw fills every kGatherWarps-th A stage (lane
    // owns rows lane, lane+32, lane+64, lane+96), so kGatherWarps stages are in
    // flight at once (each warp's cp.async batch completes in ~0.7-2 us).
    const int gw = warp - 4;
    const uint8_t* x = static_cast<const uint8_t*>(loc_ptr(d.x, p));
    const __nv_bfloat16* xb = reinterpret_cast<const __nv_bfloat16*>(x);
    const int cpt = d.Cin / 8;           // 16-byte chunks per tap (vec path)
    const int kwc = d.kw * d.Cin;        // elements per kernel row (scalar path)
    int64_t kseq = 0;                    // global A-stage counter
    for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x) {
      int hb[4], wb[4];
      int64_t img[4];
      bool mv[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int64_t m = (int64_t)tile * 128 + lane + 32 * i;
        mv[i] = m < d.npix;
        const int n = mv[i] ? (int)(m / hw) : 0;
        const int rem = mv[i] ? (int)(m % hw) : 0;
        hb[i] = (rem / d.Wo) * d.sh - d.ph;
        wb[i] = (rem % d.Wo) * d.sw - d.pw;
        img[i] = (int64_t)n * d.H * d.W;
      }
      for (int kb = 0; kb < d.katoms; ++kb, ++kseq) {
        if ((int)(kseq % kGatherWarps) != gw) continue;
        const int stage = (int)(kseq % S);
        const uint32_t phase = (uint32_t)((kseq / S) & 1);
        mbar_wait(&empty[stage], phase ^ 1);
        if (d.vec) {
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const int row = lane + 32 * i;
            uint8_t* dst = ring + stage * 16384 + row * 128;
#pragma unroll
            for (int q = 0; q < 8; ++q) {
              const int kc = kb * 8 + q;
              const uint8_t* src = x;
              uint32_t bytes = 0;
              if (mv[i] && kc < d.kchunks) {
                const int tap = kc / cpt, cc = kc - tap * cpt;
                const int hi = hb[i] + tap / d.kw, wi = wb[i] + tap % d.kw;
                if (hi >= 0 && hi < d.H && wi >= 0 && wi < d.W) {
                  src = x + ((img[i] + (int64_t)hi * d.W + wi) * d.Cin + cc * 8) * 2;
                  bytes = 16;
                }
              }
              cp_async16(dst + ((q ^ (row & 7)) * 16), src, bytes);
            }
          }
          cp_async_arrive(&full[stage]);
        } else {
          // small Cin (the 3-channel image): element gather with carried
          // (a, b, c) counters -- k = (a * kw + b) * Cin + c, no divisions
#pragma unroll 1
          for (int i = 0; i < 4; ++i) {
            const int row = lane + 32 * i;
            uint8_t* dst = ring + stage * 16384 + row * 128;
            int k = kb * 64;
            int a = k / kwc, rr = k - a * kwc;
            int b = rr / d.Cin, c = rr - b * d.Cin;
#pragma unroll 1
            for (int q = 0; q < 8; ++q) {
              uint32_t pk[4];
#pragma unroll
              for (int e2 = 0; e2 < 4; ++e2) {
                float f[2];
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                  f[h] = 0.f;
                  const int hi = hb[i] + a, wi = wb[i] + b;
                  if (mv[i] && k < d.K && hi >= 0 && hi < d.H && wi >= 0 && wi < d.W)
                    f[h] = __bfloat162float(xb[(img[i] + (int64_t)hi * d.W + wi) * d.Cin + c]);
                  ++k;
                  if (++c == d.Cin) {
                    c = 0;
                    if (++b == d.kw) b = 0, ++a;
                  }
                }
                pk[e2] = pack_bf16(f[0], f[1]);
              }
              *reinterpret_cast<uint4*>(dst + ((q ^ (row & 7)) * 16)) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
            }
          }
          fence_proxy_async();
          mbar_arrive(&full[stage]);
        }
      }
    }
  } else if (warp == 4 + kGatherWarps) {
    // ------------------------------------------------------------ weights + MMA issuer
    if (lane == 0) {
      mbar_expect_tx(wbar, wbytes);
      for (int kb = 0; kb < d.katoms; ++kb) tma_load_2d(wres + kb * d.Np * 128, d.wmap, wbar, kb * 64, blockIdx.y * d.Np);
      mbar_wait(wbar, 0);
      int stage = 0;
      uint32_t phase = 0;
      const uint32_t id = idesc_bf16(128, d.Np);
      int it = 0;
      for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x, ++it) {
        const int buf = it & 1;
        mbar_wait(&acc_empty[buf], ((it >> 1) & 1) ^ 1);
        tc_fence_after();
        const uint32_t tacc = tbase + buf * d.Np;
        for (int kb = 0; kb < d.katoms; ++kb) {
          mbar_wait(&full[stage], phase);
          fence_proxy_async();
          tc_fence_after();
          const uint32_t sa = smem_u32(ring + stage * 16384);
          const uint32_t sb = smem_u32(wres + kb * d.Np * 128);
          const int nk = min(4, (d.K - kb * 64 + 15) / 16);
          for (int k = 0; k < nk; ++k)
            mma_bf16(tacc, umma_desc(sa + 32 * k), umma_desc(sb + 32 * k), id, (kb | k) ? 1u : 0u);
          mma_commit(&empty[stage]);
          if (++stage == S) stage = 0, phase ^= 1;
        }
        mma_commit(&acc_full[buf]);
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue
    const int row = threadIdx.x;
    const uint32_t lane_off = (uint32_t)(warp * 32) << 16;
    __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.arena + d.y.off);
    const int oc0 = blockIdx.y * d.Nsl;
    int it = 0;
    for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x, ++it) {
      const int buf = it & 1;
      mbar_wait(&acc_full[buf], (it >> 1) & 1);
      tc_fence_after();
      const int64_t m = (int64_t)tile * 128 + row;
      for (int g = 0; g < d.Np / 8; ++g) {
        uint32_t v[8];
        tmem_ld8(tbase + lane_off + buf * d.Np + g * 8, v);
        tmem_wait_ld();
        const int o = oc0 + g * 8;
        if (m < d.npix && g * 8 < d.Nsl && o < d.Nout) {
          float f[8];
#pragma unroll
          for (int i = 0; i < 8; ++i) f[i] = __uint_as_float(v[i]) + (d.b >= 0 ? __ldg(p.params + d.b + o + i) : 0.f);
          *reinterpret_cast<uint4*>(y + m * d.Nout + o) =
              make_uint4(pack_bf16(f[0], f[1]), pack_bf16(f[2], f[3]), pack_bf16(f[4], f[5]), pack_bf16(f[6], f[7]));
        }
      }
      tc_fence_before();
      warp_arrive(&acc_empty[buf]);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tbase), "r"(d.tmem_cols));
  }
}


// TMA mode: 6 warps -- 0-3 epilogue, 4 TMA producer (weights once, then one
// tap-shifted strided box per (tap, 64-channel atom)), 5 MMA issuer.
constexpr int kConvTmaThreads = 192;

__global__ void __launch_bounds__(kConvTmaThreads, 1) conv_tma_kernel(const __grid_constant__ ConvTcDesc d, RunPtrs p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  const int S = d.stages;
  const int wbytes = d.katoms * d.Np * 128;
  uint8_t* wres = smem;
  uint8_t* ring = smem + wbytes;
  uint64_t* bars = reinterpret_cast<uint64_t*>(ring + S * 16384);
  uint64_t* full = bars;
  uint64_t* empty = bars + S;
  uint64_t* acc_full = bars + 2 * S;
  uint64_t* acc_empty = acc_full + 2;
  uint64_t* wbar = acc_empty + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(wbar + 1);
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&acc_full[b], 1);
      mbar_init(&acc_empty[b], 4);
    }
    mbar_init(wbar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(d.tmem_cols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tmem_slot;
  pdl_wait();
  pdl_trigger_early();
  const int per_img = d.nhb * d.nwb;

  if (warp == 4) {
    if (lane == 0) {
      mbar_expect_tx(wbar, wbytes);
      for (int kb = 0; kb < d.katoms; ++kb) tma_load_2d(wres + kb * d.Np * 128, d.wmap, wbar, kb * 64, blockIdx.y * d.Np);
      int stage = 0;
      uint32_t phase = 0;
      const uint32_t bytes = 128u * d.tw * d.th * d.tn;
      for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x) {
        const int nb = tile / per_img, rem = tile % per_img;
        const int n0 = nb * d.tn, h0 = (rem / d.nwb) * d.th, w0 = (rem % d.nwb) * d.tw;
        for (int tap = 0; tap < d.taps; ++tap) {
          const int a = tap / d.kw, b = tap % d.kw;
          for (int kc = 0; kc < d.kpt; ++kc) {
            mbar_wait(&empty[stage], phase ^ 1);
            mbar_expect_tx(&full[stage], bytes);
            tma_load_4d(ring + stage * 16384, d.xmap, &full[stage], kc * 64, w0 * d.s - d.pw + b, h0 * d.s - d.ph + a, n0);
            if (++stage == S) stage = 0, phase ^= 1;
          }
        }
      }
    }
  } else if (warp == 5) {
    if (lane == 0) {
      mbar_wait(wbar, 0);
      int stage = 0;
      uint32_t phase = 0;
      const uint32_t id = idesc_bf16(128, d.Np);
      int it = 0;
      for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x, ++it) {
        const int buf = it & 1;
        mbar_wait(&acc_empty[buf], ((it >> 1) & 1) ^ 1);
        tc_fence_after();
        const uint32_t tacc = tbase + buf * d.Np;
        for (int tap = 0; tap < d.taps; ++tap)
          for (int kc = 0; kc < d.kpt; ++kc) {
            mbar_wait(&full[stage], phase);
            tc_fence_after();
            const uint32_t sa = smem_u32(ring + stage * 16384);
            const uint32_t sb = smem_u32(wres + (tap * d.kpt + kc) * d.Np * 128);
            const int nk = min(4, (d.Cin - kc * 64 + 15) / 16);
            for (int k = 0; k < nk; ++k)
              mma_bf16(tacc, umma_desc(sa + 32 * k), umma_desc(sb + 32 * k), id, (tap | kc | k) ? 1u : 0u);
            mma_commit(&empty[stage]);
            if (++stage == S) stage = 0, phase ^= 1;
          }
        mma_commit(&acc_full[buf]);
      }
    }
  } else {
    const int row = threadIdx.x;
    const uint32_t lane_off = (uint32_t)(warp * 32) << 16;
    __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.arena + d.y.off);
    const int oc0 = blockIdx.y * d.Nsl;
    const int wi = row % d.tw, hi = (row / d.tw) % d.th, ni = row / (d.tw * d.th);
    int it = 0;
    for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x, ++it) {
      const int buf = it & 1;
      const int nb = tile / per_img, rem = tile % per_img;
      const int n = nb * d.tn + ni, ho = (rem / d.nwb) * d.th + hi, wo = (rem % d.nwb) * d.tw + wi;
      const bool valid = row < d.mused && n < d.N && ho < d.Ho && wo < d.Wo;
      const int64_t m = ((int64_t)n * d.Ho + ho) * d.Wo + wo;
      mbar_wait(&acc_full[buf], (it >> 1) & 1);
      tc_fence_after();
      for (int g = 0; g < d.Np / 8; ++g) {
        uint32_t v[8];
        tmem_ld8(tbase + lane_off + buf * d.Np + g * 8, v);
        tmem_wait_ld();
        const int o = oc0 + g * 8;
        if (valid && g * 8 < d.Nsl && o < d.Nout) {
          float f[8];
#pragma unroll
          for (int i = 0; i < 8; ++i) f[i] = __uint_as_float(v[i]) + (d.b >= 0 ? __ldg(p.params + d.b + o + i) : 0.f);
          *reinterpret_cast<uint4*>(y + m * d.Nout + o) =
              make_uint4(pack_bf16(f[0], f[1]), pack_bf16(f[2], f[3]), pack_bf16(f[4], f[5]), pack_bf16(f[6], f[7]));
        }
      }
      tc_fence_before();
      warp_arrive(&acc_empty[buf]);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tbase), "r"(d.tmem_cols));
  }
}

}  // namespace

void launch_conv_tc(const ConvTcDesc& d, const RunPtrs& p, cudaStream_t s) {
  static bool configured = false;
  static int sms = 0;
  if (!configured) {
    cudaFuncSetAttribute(conv_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    cudaFuncSetAttribute(conv_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    configured = true;
  }
  // persistent, one CTA per SM, output-channel slices along y
  const int grid = std::min(d.ntiles, std::max(1, (sms > 0 ? sms : 148) / d.nsl));
  if (d.tma)
    launch_pdl(conv_tma_kernel, dim3(grid, d.nsl), dim3(kConvTmaThreads), std::max(d.smem_bytes, 116 * 1024), s, d, p);
  else
    conv_tc_kernel<<<dim3(grid, d.nsl), kConvThreads, std::max(d.smem_bytes, 116 * 1024), s>>>(d, p);
}

}  // namespace temco
