// Reduced-rank core convolution on tensor cores (bf16 mode): the Tucker core
// K x K conv R_in -> R_out (and its 1x1 / strided variants, the downsample
// cores), Eq. (2) P:L106 -- SURVEY 8(a) row a7.
//
// These convs are HBM-bound (R_in, R_out = 8..208, AI ~ 25 flop/B): the job
// is to stream the reduced input once and write the reduced output once.
// Implicit GEMM with mma.sync m16n8k16: a warp owns 16 output pixels at a
// time and walks its (block, tap) units; the A fragments of a unit are
// gathered straight from global memory into registers (the tap-shifted NHWC
// rows, 32-bit loads, zero outside the image) with the next two units' loads
// in flight; the weights [tap][R_out][R_in] are ldmatrix'd from SMEM; fp32
// accumulation over taps and channels; bf16 NHWC output from the fragments.
#include <cuda_bf16.h>

#include <algorithm>

#include "kernels.h"

namespace temco {

namespace {

constexpr int kRkWarps = 16;

__device__ __forceinline__ uint32_t s_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void ldsm_x4(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0, %1, %2, %3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}

__device__ __forceinline__ void ldsm_x2(uint32_t addr, uint32_t& r0, uint32_t& r1) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x2.shared.b16 {%0, %1}, [%2];" : "=r"(r0), "=r"(r1) : "r"(addr));
}

__device__ __forceinline__ void mma16816(float (&c)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0, %1, %2, %3}, {%4, %5, %6, %7}, {%8, %9}, "
      "{%0, %1, %2, %3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

__device__ __forceinline__ uint32_t pk2(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}

__device__ __forceinline__ bool all_taps_mode(const RankConvDesc& d) { return d.all_taps != 0; }

struct RkCursor {
  int blk, tap, kc, nc;          // block, tap, 64-channel input chunk, 64-channel output chunk
  int hi0[2], wi0[2], nrow[2];   // per fragment row: window origin, n * H
  bool ok[2];                    // output row exists
};

__device__ __forceinline__ void rk_set_block(const RankConvDesc& d, RkCursor& u, int g) {
  const int hw = d.Ho * d.Wo;
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    const int m = u.blk * 16 + g + 8 * h;
    const int n = m / hw, rem = m - n * hw;
    const int ho = rem / d.Wo, wo = rem - ho * d.Wo;
    u.hi0[h] = ho * d.sh - d.ph;
    u.wi0[h] = wo * d.sw - d.pw;
    u.nrow[h] = n * d.H;
    u.ok[h] = m < d.npix;
  }
}

// tap-shifted NHWC row pair of one tap: 32-bit word offsets, validity
__device__ __forceinline__ void rk_rows(const RankConvDesc& d, const RkCursor& u, int tap, int64_t (&p)[2],
                                        bool (&v)[2]) {
  const int ty = tap / d.kw, tx = tap - ty * d.kw;
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    const int hi = u.hi0[h] + ty, wi = u.wi0[h] + tx;
    v[h] = u.ok[h] && tap < d.kh * d.kw && hi >= 0 && hi < d.H && wi >= 0 && wi < d.W;
    p[h] = ((int64_t)(u.nrow[h] + hi) * d.W + wi) * (d.C / 2);
  }
}

template <int KS>
__device__ __forceinline__ void rk_load(uint32_t (&a)[KS][4], const RankConvDesc& d, const uint32_t* __restrict__ x,
                                        const RkCursor& u, int t4) {
  if (d.pair) {
    // Cin == 8: one k-step holds two taps (k 0-7: tap 2u, k 8-15: tap 2u + 1)
    int64_t p0[2], p1[2];
    bool v0[2], v1[2];
    rk_rows(d, u, 2 * u.tap, p0, v0);
    rk_rows(d, u, 2 * u.tap + 1, p1, v1);
    a[0][0] = v0[0] ? __ldg(x + p0[0] + t4) : 0u;
    a[0][1] = v0[1] ? __ldg(x + p0[1] + t4) : 0u;
    a[0][2] = v1[0] ? __ldg(x + p1[0] + t4) : 0u;
    a[0][3] = v1[1] ? __ldg(x + p1[1] + t4) : 0u;
    return;
  }
  const int ty = u.tap / d.kw, tx = u.tap - ty * d.kw;
  int64_t p[2];
  bool v[2];
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    const int hi = u.hi0[h] + ty, wi = u.wi0[h] + tx;
    v[h] = u.ok[h] && hi >= 0 && hi < d.H && wi >= 0 && wi < d.W;
    p[h] = ((int64_t)(u.nrow[h] + hi) * d.W + wi) * (d.C / 2);
  }
#pragma unroll
  for (int ks = 0; ks < KS; ++ks) {
    const int k0 = u.kc * 64 + ks * 16 + 2 * t4, k1 = k0 + 8;
    a[ks][0] = (v[0] && k0 < d.C) ? __ldg(x + p[0] + k0 / 2) : 0u;
    a[ks][1] = (v[1] && k0 < d.C) ? __ldg(x + p[1] + k0 / 2) : 0u;
    a[ks][2] = (v[0] && k1 < d.C) ? __ldg(x + p[0] + k1 / 2) : 0u;
    a[ks][3] = (v[1] && k1 < d.C) ? __ldg(x + p[1] + k1 / 2) : 0u;
  }
}

template <int KS, int NT, bool KCH>   // KCH: Cin > 64, walk 64-channel input chunks
__global__ void __launch_bounds__(32 * kRkWarps, 1) conv_rank_mma_kernel(const __grid_constant__ RankConvDesc d,
                                                                         RunPtrs p, const uint16_t* __restrict__ tcw) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int g = lane / 4, t4 = lane % 4;
  {
    const uint4* src = reinterpret_cast<const uint4*>(tcw + d.wblob);
    uint4* dst = reinterpret_cast<uint4*>(smem);
    for (int i = threadIdx.x; i < d.blob_bytes / 16; i += blockDim.x) dst[i] = __ldg(src + i);
  }
  __syncthreads();
  pdl_wait();
  pdl_trigger_early();
  const __nv_bfloat16* wb = reinterpret_cast<const __nv_bfloat16*>(smem);
  const uint32_t* x = reinterpret_cast<const uint32_t*>(loc_ptr(d.x, p));
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(const_cast<void*>(loc_ptr(d.y, p)));
  const int taps = d.pair ? (d.kh * d.kw + 1) / 2 : d.kh * d.kw;   // units per block
  const int ws = d.wstride;                       // elements per weight row (C padded + 8)
  // ldmatrix lane addressing: x4 = (n-tile + q / 2, k half q % 2); x2 = (n-tile, k half q % 2)
  const int lq = lane >> 3, lr = lane & 7;
  const uint32_t wbase4 = s_u32(wb + ((lq >> 1) * 8 + lr) * ws + (lq & 1) * 8);
  const uint32_t wbase2 = s_u32(wb + lr * ws + (lq & 1) * 8);
  const int nw = gridDim.x * kRkWarps;
  if constexpr (KS <= 2 && !KCH) {
    if ((d.nblocks <= 2 * nw || all_taps_mode(d)) && taps <= 9) {
      // every tap's A fragments of the block in flight at once (instead of two units ahead)
      for (int blk = blockIdx.x * kRkWarps + warp; blk < d.nblocks; blk += nw) {
        RkCursor u{};
        u.blk = blk;
        rk_set_block(d, u, g);
        uint32_t at[9][KS][4];
#pragma unroll
        for (int t = 0; t < 9; ++t) {
          u.tap = t;
          if (t < taps) rk_load<KS>(at[t], d, x, u, t4);
        }
        float acc[NT][4];
#pragma unroll
        for (int nt = 0; nt < NT; ++nt) {
          float b0 = 0.f, b1 = 0.f;
          if (d.b >= 0) {
            b0 = p.params[d.b + nt * 8 + 2 * t4];
            b1 = p.params[d.b + nt * 8 + 2 * t4 + 1];
          }
          acc[nt][0] = acc[nt][2] = b0;
          acc[nt][1] = acc[nt][3] = b1;
        }
#pragma unroll
        for (int t = 0; t < 9; ++t) {
          if (t >= taps) break;
          const uint32_t tw = (uint32_t)(t * d.K * ws * 2);
#pragma unroll
          for (int ks = 0; ks < KS; ++ks) {
#pragma unroll
            for (int np = 0; np < NT / 2; ++np) {
              uint32_t b0, b1, b2, b3;
              ldsm_x4(wbase4 + tw + (uint32_t)((np * 16 * ws + ks * 16) * 2), b0, b1, b2, b3);
              mma16816(acc[2 * np], at[t][ks], b0, b1);
              mma16816(acc[2 * np + 1], at[t][ks], b2, b3);
            }
            if (NT & 1) {
              uint32_t b0, b1;
              ldsm_x2(wbase2 + tw + (uint32_t)(((NT - 1) * 8 * ws + ks * 16) * 2), b0, b1);
              mma16816(acc[NT - 1], at[t][ks], b0, b1);
            }
          }
        }
        const int m0 = blk * 16 + g, m1 = m0 + 8;
#pragma unroll
        for (int nt = 0; nt < NT; ++nt) {
          const int col = nt * 8 + 2 * t4;
          if (m0 < d.npix) *reinterpret_cast<uint32_t*>(y + (int64_t)m0 * d.K + col) = pk2(acc[nt][0], acc[nt][1]);
          if (m1 < d.npix) *reinterpret_cast<uint32_t*>(y + (int64_t)m1 * d.K + col) = pk2(acc[nt][2], acc[nt][3]);
        }
      }
      return;
    }
  }
  // unit order per block: output chunk, tap, input chunk
  auto advance = [&](RkCursor& u) {
    if (KCH && ++u.kc < d.nkc) return;
    u.kc = 0;
    if (++u.tap < taps) return;
    u.tap = 0;
    u.blk += nw;
    if (u.blk < d.nblocks) rk_set_block(d, u, g);
  };
  RkCursor cur{};
  cur.blk = blockIdx.x * kRkWarps + warp;
  if (cur.blk < d.nblocks) rk_set_block(d, cur, g);
  RkCursor pf = cur;
  uint32_t a[KS][4], an[KS][4], ann[KS][4];
  if (pf.blk < d.nblocks) rk_load<KS>(a, d, x, pf, t4);
  advance(pf);
  if (pf.blk < d.nblocks) rk_load<KS>(an, d, x, pf, t4);
  advance(pf);
  float acc[NT][4];
  for (; cur.blk < d.nblocks; advance(cur)) {
    if (pf.blk < d.nblocks) rk_load<KS>(ann, d, x, pf, t4);
    advance(pf);
    constexpr int ntc = NT;                            // K <= 64: one output chunk
    if (cur.tap == 0 && cur.kc == 0) {
#pragma unroll
      for (int nt = 0; nt < NT; ++nt) {
        float b0 = 0.f, b1 = 0.f;
        if (d.b >= 0 && nt < ntc) {
          b0 = p.params[d.b + nt * 8 + 2 * t4];
          b1 = p.params[d.b + nt * 8 + 2 * t4 + 1];
        }
        acc[nt][0] = acc[nt][2] = b0;
        acc[nt][1] = acc[nt][3] = b1;
      }
    }
    const uint32_t tw = (uint32_t)((cur.tap * d.K * ws + (KCH ? cur.kc * 64 : 0)) * 2);
#pragma unroll
    for (int ks = 0; ks < KS; ++ks) {
      if (KCH && cur.kc * 64 + ks * 16 >= d.C) break;      // the last input chunk may be short
#pragma unroll
      for (int np = 0; np < NT / 2; ++np) {
        if (2 * np + 1 < ntc) {
          uint32_t b0, b1, b2, b3;
          ldsm_x4(wbase4 + tw + (uint32_t)((np * 16 * ws + ks * 16) * 2), b0, b1, b2, b3);
          mma16816(acc[2 * np], a[ks], b0, b1);
          mma16816(acc[2 * np + 1], a[ks], b2, b3);
        } else if (2 * np < ntc) {
          uint32_t b0, b1;
          ldsm_x2(wbase2 + tw + (uint32_t)((2 * np * 8 * ws + ks * 16) * 2), b0, b1);
          mma16816(acc[2 * np], a[ks], b0, b1);
        }
      }
      if ((NT & 1) && NT - 1 < ntc) {
        uint32_t b0, b1;
        ldsm_x2(wbase2 + tw + (uint32_t)(((NT - 1) * 8 * ws + ks * 16) * 2), b0, b1);
        mma16816(acc[NT - 1], a[ks], b0, b1);
      }
    }
    if (cur.tap == taps - 1 && (!KCH || cur.kc == d.nkc - 1)) {
      const int m0 = cur.blk * 16 + g, m1 = m0 + 8;
#pragma unroll
      for (int nt = 0; nt < NT; ++nt) {
        const int col = nt * 8 + 2 * t4;
        if (m0 < d.npix) *reinterpret_cast<uint32_t*>(y + (int64_t)m0 * d.K + col) = pk2(acc[nt][0], acc[nt][1]);
        if (m1 < d.npix) *reinterpret_cast<uint32_t*>(y + (int64_t)m1 * d.K + col) = pk2(acc[nt][2], acc[nt][3]);
      }
    }
#pragma unroll
    for (int ks = 0; ks < KS; ++ks)
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        a[ks][i] = an[ks][i];
        an[ks][i] = ann[ks][i];
      }
  }
}

template <int KS, int NT, bool KCH>
void launch_rk_t(const RankConvDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  static bool configured = false;
  static int sms = 148;
  if (!configured) {
    cudaFuncSetAttribute(conv_rank_mma_kernel<KS, NT, KCH>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    configured = true;
  }
  const int grid = std::min((d.nblocks + kRkWarps - 1) / kRkWarps, sms);
  launch_pdl(conv_rank_mma_kernel<KS, NT, KCH>, dim3(grid), dim3(32 * kRkWarps), d.blob_bytes, s, d, p, tcw);
}

uint16_t f2bf(float f) {
  uint32_t u;
  memcpy(&u, &f, 4);
  u += 0x7FFF + ((u >> 16) & 1);
  return (uint16_t)(u >> 16);
}

}  // namespace

bool conv_rank_mma_lower(const ConvDesc& c, const float* w_khkwc, std::vector<uint16_t>& tcw, RankConvDesc& d) {
  if (c.groups != 1 || c.x.dtype != DT_BF16 || c.y.dtype != DT_BF16 || c.C % 8 || c.K % 8) return false;
  // up to 64 input / output channels per unit; wider convs walk 64-channel chunks
  const int nkc = (c.C + 63) / 64, nnc = (c.K + 63) / 64;
  const int KS = nkc > 1 ? 4 : (c.C + 15) / 16, NT = c.K / 8;
  if (nkc * 64 > 256 || nnc > 1 || (int64_t)c.N * c.Ho * c.Wo >= (1LL << 31) - 16) return false;
  d = RankConvDesc();
  d.x = c.x;
  d.y = c.y;
  d.N = c.N; d.H = c.H; d.W = c.W; d.C = c.C;
  d.Ho = c.Ho; d.Wo = c.Wo; d.K = c.K;
  d.kh = c.kh; d.kw = c.kw; d.sh = c.sh; d.sw = c.sw; d.ph = c.ph; d.pw = c.pw;
  d.b = c.b;
  d.npix = c.N * c.Ho * c.Wo;
  d.nblocks = (d.npix + 15) / 16;
  d.KS = KS;
  d.NT = NT;
  d.nkc = nkc;
  d.nnc = nnc;
  // weights [tap][K][KS*16 + 8] bf16 (row stride an odd number of 16-byte chunks:
  // conflict-free ldmatrix), zero K padding
  d.wstride = (nkc > 1 ? nkc * 64 : KS * 16) + 8;
  const int taps = c.kh * c.kw;
  d.pair = (c.C == 8 && taps > 1 && nkc == 1) ? 1 : 0;
  // all taps of a block in flight at once (measured better than the two-units-ahead walk for
  // single-k-step convs: DenseNet's 3x3 cores -8 %, ResNet-50's -4 %)
  d.all_taps = getenv("TEMCO_RK_TWO_AHEAD") ? 0 : 1;
  const int units = d.pair ? (taps + 1) / 2 : taps;
  std::vector<uint16_t> blob((size_t)units * c.K * d.wstride, 0);
  for (int t = 0; t < taps; ++t) {
    const int u = d.pair ? t / 2 : t, k0 = d.pair ? (t % 2) * 8 : 0;
    for (int k = 0; k < c.K; ++k)
      for (int ci = 0; ci < c.C; ++ci)
        blob[((size_t)u * c.K + k) * d.wstride + k0 + ci] = f2bf(w_khkwc[((size_t)k * taps + t) * c.C + ci]);
  }
  d.blob_bytes = (int)((blob.size() * 2 + 15) / 16 * 16);
  if (d.blob_bytes > 200 * 1024) return false;
  while (tcw.size() % 512) tcw.push_back(0);
  d.wblob = (int64_t)tcw.size();
  tcw.insert(tcw.end(), blob.begin(), blob.end());
  while (tcw.size() % 8) tcw.push_back(0);
  d.alg_flops = 2LL * d.npix * c.K * c.C * taps;
  d.alg_bytes = 2LL * ((int64_t)c.N * c.H * c.W * c.C + (int64_t)d.npix * c.K);
  return true;
}

void launch_conv_rank_mma(const RankConvDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
#define TEMCO_RK_CASE(ks, nt) \
  if (d.nkc == 1 && d.KS == ks && d.NT == nt) return launch_rk_t<ks, nt, false>(d, tcw, p, s); \
  if (d.nkc > 1 && ks == 4 && d.NT == nt) return launch_rk_t<4, nt, true>(d, tcw, p, s);
#define TEMCO_RK_ROW(ks) \
  TEMCO_RK_CASE(ks, 1) TEMCO_RK_CASE(ks, 2) TEMCO_RK_CASE(ks, 3) TEMCO_RK_CASE(ks, 4) \
  TEMCO_RK_CASE(ks, 5) TEMCO_RK_CASE(ks, 6) TEMCO_RK_CASE(ks, 7) TEMCO_RK_CASE(ks, 8)
  TEMCO_RK_ROW(1) TEMCO_RK_ROW(2) TEMCO_RK_ROW(3) TEMCO_RK_ROW(4)
#undef TEMCO_RK_ROW
#undef TEMCO_RK_CASE
}

}  // namespace temco
