// TMA-staged reduced-rank core convolution (sm_100a): see tile.h.
//
// Per CTA (8 warps, persistent over output tiles of TN images x TH rows x TW columns):
//   * one thread issues the 4-D TMA box (C, FW, FH, TN) of tile i + 2 into the buffer tile i
//     just released: two footprints in flight, the zero padding of the conv comes from the
//     TMA's out-of-bounds fill.  Pixel rows of 32 / 64 / 128 bytes (C = 16 / 32 / 64) are
//     TMA-swizzled so that the 8 rows of an ldmatrix land in 8 different bank groups; C = 8,
//     56, 104 (an odd number of 16-byte chunks per pixel) are conflict-free unswizzled.
//   * a warp computes two m-tiles of 16 output pixels: for every k-step (a tap x 16 input
//     channels, or for C = 8 two taps x 8 channels) one ldmatrix.x4 per m-tile gathers the A
//     fragment (lane = pixel row; the tap shift is an address offset into the footprint) and
//     one ldmatrix.x4 per pair of n-tiles the B fragments (weights [k-step][k half][n][8],
//     8 consecutive 16-byte rows: conflict-free), shared by both m-tiles.
//   * fp32 accumulation (+ bias), bf16 NHWC stores from the fragments.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cudaTypedefs.h>

#include <algorithm>

#include "tmap.h"
#include "tc_ptx.cuh"
#include "tile.h"

namespace temco {

namespace {

constexpr int kTcWarps = 8, kTcThreads = 32 * (kTcWarps + 1);   // + the TMA producer warp
constexpr int kTcBufs = 3;                                             // footprints in flight
constexpr int kTcFootBudget = 32 * 1024;   // bytes of one footprint buffer (three in flight, 2 CTAs / SM)

uint16_t f2bf_t(float f) {
  uint32_t u;
  memcpy(&u, &f, 4);
  u += 0x7FFF + ((u >> 16) & 1);
  return (uint16_t)(u >> 16);
}

}  // namespace

bool tile_conv_lower(const ConvDesc& c, const float* w, std::vector<uint16_t>& tcw, TileConvDesc& d) {
  if (getenv("TEMCO_NO_TILECONV")) return false;
  if (c.groups != 1 || c.x.dtype != DT_BF16 || c.y.dtype != DT_BF16 || c.C % 8 || c.K % 8 || c.K > 64) return false;
  if (c.x.where != W_ARENA || c.C > 104 || c.kh > 7 || c.kw > 7) return false;
  d = TileConvDesc();
  d.x = c.x;
  d.y = c.y;
  d.N = c.N; d.H = c.H; d.W = c.W; d.C = c.C;
  d.Ho = c.Ho; d.Wo = c.Wo; d.K = c.K;
  d.kh = c.kh; d.kw = c.kw; d.sh = c.sh; d.sw = c.sw; d.ph = c.ph; d.pw = c.pw;
  d.b = c.b;
  d.dbg = getenv("TEMCO_TILE_DBG") ? atoi(getenv("TEMCO_TILE_DBG")) : 0;
  const int taps = c.kh * c.kw;
  d.pair = (c.C == 8 && taps > 1) ? 1 : 0;
  d.ksc = (c.C + 15) / 16;
  d.nks = d.pair ? (taps + 1) / 2 : taps * d.ksc;
  const int cb = c.C * 2;
  // 1x1 strided cores (the downsample cores): the TMA box takes every sh-th row / sw-th column
  const bool sub = c.kh == 1 && c.kw == 1;
  // TMA view: cw pixels per inner row (up to 128 bytes) so that narrow pixels (C = 8 .. 32) are not
  // fetched 16 / 32 / 64 bytes per TMA row; the inner row is the swizzle span
  d.cw = 1;
  if (!sub)
    while (d.cw * 2 * cb <= 128 && c.W % (d.cw * 2) == 0) d.cw *= 2;
  const int ib = d.cw * cb;
  d.swz = ib == 32 ? 1 : ib == 64 ? 2 : ib == 128 ? 3 : 0;
  // tile: columns split into <= 32-wide equal parts; whole small images grouped
  const int ntw = (c.Wo + 31) / 32;
  d.TW = (c.Wo + ntw - 1) / ntw;
  d.TN = 1;
  if (c.Ho * d.TW < 128) d.TN = std::max(1, std::min({c.N, 256 / (c.Ho * d.TW), 256}));
  d.TH = d.TN > 1 ? c.Ho : std::min(c.Ho, (256 + d.TW - 1) / d.TW);
  auto foot = [&](int TH, int TN) {   // TMA bytes of a footprint: FH rows of G inner rows
    const int FH = sub ? TH : (TH - 1) * c.sh + c.kh, FW = sub ? d.TW : (d.TW - 1) * c.sw + c.kw;
    const int G = (FW + d.cw - 1 + d.cw - 1) / d.cw;   // any start offset within an inner row
    return (int64_t)FH * (sub ? FW : G * d.cw) * TN * cb;
  };
  while (d.TN > 1 && foot(d.TH, d.TN) > kTcFootBudget) --d.TN;
  while (d.TH > 1 && foot(d.TH, d.TN) > kTcFootBudget) --d.TH;
  if (foot(d.TH, d.TN) > kTcFootBudget) return false;
  d.FH = sub ? d.TH : (d.TH - 1) * c.sh + c.kh;
  d.FW = sub ? d.TW : (d.TW - 1) * c.sw + c.kw;
  if (d.FW > 256 || d.FH > 256 || (sub ? std::max(d.TW * c.sw, d.TH * c.sh) > 256 : false)) return false;
  // enough tiles for two CTAs per SM where the tensor allows: fewer images, then fewer rows
  auto count = [&](int TH, int TN) {
    return (int64_t)((c.Wo + d.TW - 1) / d.TW) * ((c.Ho + TH - 1) / TH) * ((c.N + TN - 1) / TN);
  };
  while (d.TN > 1 && count(d.TH, d.TN) < 296) d.TN = (d.TN + 1) / 2;
  while (d.TN == 1 && d.TH * d.TW > 64 && d.TH > 1 && count(d.TH, 1) < 296) d.TH = (d.TH + 1) / 2;
  d.FH = sub ? d.TH : (d.TH - 1) * c.sh + c.kh;
  d.FW = sub ? d.TW : (d.TW - 1) * c.sw + c.kw;
  d.G = sub ? d.FW : (d.FW + 2 * d.cw - 2) / d.cw;
  d.RP = sub ? d.FW : d.G * d.cw;
  if (d.G > 256) return false;
  d.tiles_w = (c.Wo + d.TW - 1) / d.TW;
  d.tiles_h = (c.Ho + d.TH - 1) / d.TH;
  d.tiles_n = (c.N + d.TN - 1) / d.TN;
  const int64_t nt = (int64_t)d.tiles_w * d.tiles_h * d.tiles_n;
  if (nt >= (1LL << 31)) return false;
  d.ntiles = (int)nt;
  d.box_bytes = (int)foot(d.TH, d.TN);
  d.buf_bytes = (d.box_bytes + 64 + 1023) / 1024 * 1024;   // + zeroed slack: the half k-step past C
  d.Kp = (c.K + 15) / 16 * 16;
  d.w_bytes = d.nks * 2 * d.Kp * 16;
  d.smem_bytes = 1024 + kTcBufs * d.buf_bytes + d.w_bytes + 64 + d.nks * 2 * 8 + kTcBufs * 16;
  auto magic = [](int dv, uint32_t& m, uint32_t& sh) {   // q / dv = (umulhi(q, m) + q) >> sh
    sh = 0;
    while ((1u << sh) < (uint32_t)dv) ++sh;
    m = (uint32_t)((((uint64_t)1 << 32) * ((1ull << sh) - (uint64_t)dv)) / (uint64_t)dv + 1);
  };
  magic(d.TH * d.TW, d.mpx, d.spx);
  magic(d.TW, d.mtw, d.stw);
  if (d.smem_bytes > 227 * 1024) return false;
  // weights [ks][k half][n][8]: k-step ks, k = half * 8 + j  ->  (tap, channel)
  std::vector<uint16_t> blob((size_t)d.nks * 2 * d.Kp * 8, 0);
  for (int ks = 0; ks < d.nks; ++ks)
    for (int h = 0; h < 2; ++h)
      for (int n = 0; n < c.K; ++n)
        for (int j = 0; j < 8; ++j) {
          int tap, ch;
          if (d.pair) {
            tap = 2 * ks + h;
            ch = j;
          } else {
            tap = ks / d.ksc;
            ch = (ks % d.ksc) * 16 + h * 8 + j;
          }
          if (tap >= taps || ch >= c.C) continue;
          blob[(((size_t)ks * 2 + h) * d.Kp + n) * 8 + j] = f2bf_t(w[((size_t)n * taps + tap) * c.C + ch]);
        }
  while (tcw.size() % 512) tcw.push_back(0);
  d.wblob = (int64_t)tcw.size();
  tcw.insert(tcw.end(), blob.begin(), blob.end());
  const int64_t npix = (int64_t)c.N * c.Ho * c.Wo;
  d.alg_flops = npix * 2LL * c.K * c.C * taps;
  d.alg_bytes = (int64_t)c.N * c.H * c.W * cb + npix * c.K * 2;
  return true;
}

bool tile_conv_finalize(TileConvDesc& d, const char* arena, std::string& err) {
  const auto encode = tmap_encoder(err);
  if (!encode) return false;
  const bool sub = d.kh == 1 && d.kw == 1;
  // view (cw * C, W / cw, H, N): an inner row = cw consecutive pixels of an image row
  cuuint64_t dims[4] = {(cuuint64_t)d.cw * d.C, (cuuint64_t)(d.W / d.cw), (cuuint64_t)d.H, (cuuint64_t)d.N};
  cuuint64_t strides[3] = {(cuuint64_t)d.cw * d.C * 2, (cuuint64_t)d.W * d.C * 2, (cuuint64_t)d.H * d.W * d.C * 2};
  cuuint32_t box[4] = {(cuuint32_t)(d.cw * d.C), (cuuint32_t)(sub ? d.TW * d.sw : d.G),
                       (cuuint32_t)(sub ? d.TH * d.sh : d.FH), (cuuint32_t)d.TN};
  cuuint32_t es[4] = {1, (cuuint32_t)(sub ? d.sw : 1), (cuuint32_t)(sub ? d.sh : 1), 1};
  const CUtensorMapSwizzle sw = d.swz == 1   ? CU_TENSOR_MAP_SWIZZLE_32B
                                : d.swz == 2 ? CU_TENSOR_MAP_SWIZZLE_64B
                                : d.swz == 3 ? CU_TENSOR_MAP_SWIZZLE_128B
                                             : CU_TENSOR_MAP_SWIZZLE_NONE;
  CUresult r = encode(reinterpret_cast<CUtensorMap*>(d.xmap), CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4,
                      const_cast<char*>(arena + d.x.off), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
                      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    err = "cuTensorMapEncodeTiled failed (tile conv input)";
    return false;
  }
  return true;
}

namespace {
using namespace ptx;

__device__ __forceinline__ void ldsm4(uint32_t addr, uint32_t (&r)[4]) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0, %1, %2, %3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3])
               : "r"(addr));
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

// q / d for q < 2^24 by multiply-high (d >= 1): the magic pair is computed on the host
__device__ __forceinline__ int fdiv(int q, uint32_t m, uint32_t sh) {
  return (int)((__umulhi((uint32_t)q, m) + (uint32_t)q) >> sh);
}

template <int NT2, int NTU>   // pairs of n-tiles (Kp / 16); n-tiles used (K / 8: 1 for the 8-channel cores)
__global__ void __launch_bounds__(kTcThreads, NT2 >= 3 ? 1 : 2) tile_conv_kernel(const __grid_constant__ TileConvDesc d, RunPtrs p,
                                                                  const uint16_t* __restrict__ tcw) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  uint8_t* wsm = smem + kTcBufs * d.buf_bytes;
  uint64_t* full = reinterpret_cast<uint64_t*>(wsm + d.w_bytes);   // [kTcBufs] TMA bytes landed
  uint64_t* empty = full + kTcBufs;                                // [kTcBufs] the compute warps are done
  int2* ktab = reinterpret_cast<int2*>(full + 8);   // per (k-step, k half): footprint pixel offset, byte offset
  int4* tinfo = reinterpret_cast<int4*>(ktab + 2 * d.nks);   // per buffer: its tile's n0, oh0, ow0, column shift
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int g = lane >> 2, t4 = lane & 3;
  const bool sub = d.kh == 1 && d.kw == 1;
  const int she = sub ? 1 : d.sh, swe = sub ? 1 : d.sw;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kTcBufs; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], kTcWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    prefetch_tmap(d.xmap);
  }
  {
    const uint4* src = reinterpret_cast<const uint4*>(tcw + d.wblob);
    uint4* dst = reinterpret_cast<uint4*>(wsm);
    for (int i = threadIdx.x; i < d.w_bytes / 16; i += blockDim.x) dst[i] = __ldg(src + i);
    const int taps = d.kh * d.kw;
    for (int i = threadIdx.x; i < 2 * d.nks; i += blockDim.x) {
      const int ks = i >> 1, h = i & 1;
      int tap, boff;
      if (d.pair) {
        tap = min(2 * ks + h, taps - 1);   // a missing odd tap: any finite data (zero weights)
        boff = 0;
      } else {
        tap = ks / d.ksc;
        boff = (ks % d.ksc) * 32 + h * 16;
      }
      const int ty = tap / d.kw, tx = tap - ty * d.kw;
      ktab[i] = make_int2(ty * d.RP + tx, boff);
    }
    // slack after each footprint: the upper half of the last k-step of C % 16 == 8 reads 16 bytes
    // past the last pixel (zero weights; the data must only be finite)
    for (int b = 0; b < kTcBufs; ++b)
      for (int i = d.box_bytes / 16 + threadIdx.x; i < d.buf_bytes / 16; i += blockDim.x)
        reinterpret_cast<uint4*>(smem + b * d.buf_bytes)[i] = make_uint4(0, 0, 0, 0);
  }
  __syncthreads();
  pdl_wait();
  if (d.dbg & 4) return;
  const int G = gridDim.x;
  const int tpi = d.tiles_w * d.tiles_h;
  if (warp == kTcWarps) {
    // ---- producer: the footprint of this CTA's i-th tile into buffer i % kTcBufs, once the
    // compute warps released that buffer's previous tile
    if (lane == 0) {
      int it = 0;
      for (int tile = blockIdx.x; tile < d.ntiles; tile += G, ++it) {
        const int b = it % kTcBufs;
        if (it >= kTcBufs) mbar_wait(&empty[b], (uint32_t)(it / kTcBufs - 1) & 1u);
        const int tn = tile / tpi, th = (tile / d.tiles_w) % d.tiles_h, tw = tile % d.tiles_w;
        if (d.dbg & 2) {
          const int x0 = tw * d.TW * d.sw - d.pw;
          tinfo[b] = make_int4(tn * d.TN, th * d.TH, tw * d.TW, x0 - (x0 >= 0 ? x0 / d.cw : -((d.cw - 1 - x0) / d.cw)) * d.cw);
          mbar_arrive(&full[b]);
          continue;
        }
        const int x0 = tw * d.TW * d.sw - d.pw;   // first footprint column; its inner row (floor)
        const int xg = x0 >= 0 ? x0 / d.cw : -((d.cw - 1 - x0) / d.cw);
        // the tile's coordinates for the compute warps (published by the barrier's arrive: release)
        tinfo[b] = make_int4(tn * d.TN, th * d.TH, tw * d.TW, x0 - xg * d.cw);
        mbar_expect_tx(&full[b], (uint32_t)d.box_bytes);
        tma_load_4d(smem + b * d.buf_bytes, d.xmap, &full[b], 0, xg, th * d.TH * d.sh - d.ph, tn * d.TN);
      }
    }
    return;
  }
  const uint32_t wbase = smem_u32(wsm);
  const int cb = d.C * 2;
  const uint32_t smask = d.swz == 0 ? 0u : (1u << d.swz) - 1u;
  const int pxt = d.TH * d.TW, npx = d.TN * pxt, nmt = (npx + 15) / 16, npair = (nmt + 1) / 2;
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(const_cast<void*>(loc_ptr(d.y, p)));
  float bias[NTU][2];
#pragma unroll
  for (int nt = 0; nt < NTU; ++nt)
#pragma unroll
    for (int e = 0; e < 2; ++e) {
      const int col = nt * 8 + 2 * t4 + e;
      bias[nt][e] = (d.b >= 0 && col < d.K) ? p.params[d.b + col] : 0.f;
    }
  // this lane's ldmatrix row of an m-tile (A): row r of the 16, k half kh
  const int ar = (lane & 7) + ((lane >> 3) & 1) * 8, akh = lane >> 4;
  const uint32_t boff_lane = (uint32_t)(((lane >> 3) & 1) * d.Kp + (lane >> 4) * 8 + (lane & 7)) * 16u;
  int it = 0, pstart = 0;   // pairs of m-tiles are dealt round-robin over the warps ACROSS tiles
  for (int tile = blockIdx.x; tile < d.ntiles; tile += G, ++it, pstart += npair) {
    const int b = it % kTcBufs;
    mbar_wait(&full[b], (uint32_t)(it / kTcBufs) & 1u);
    const uint32_t fbase = smem_u32(smem + b * d.buf_bytes);
    const int4 ti = tinfo[b];   // written by the producer before the barrier's arrive
    const int n0 = ti.x, oh0 = ti.y, ow0 = ti.z, xr = ti.w;
    int pr = warp - pstart % kTcWarps;
    if (pr < 0) pr += kTcWarps;
    if (d.dbg & 1) pr = npair;
    for (; pr < npair; pr += kTcWarps) {
      const int mt0 = 2 * pr;
      int pbase[2];
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        int q = (mt0 + j) * 16 + ar;
        if (q >= npx) q = 0;
        const int pn = fdiv(q, d.mpx, d.spx), rem = q - pn * pxt, py = fdiv(rem, d.mtw, d.stw), px = rem - py * d.TW;
        pbase[j] = (pn * d.FH + py * she) * d.RP + px * swe + xr;   // + the box's start offset
      }
      float acc[2][NTU][4];
#pragma unroll
      for (int j = 0; j < 2; ++j)
#pragma unroll
        for (int nt = 0; nt < NTU; ++nt) {
          acc[j][nt][0] = acc[j][nt][2] = bias[nt][0];
          acc[j][nt][1] = acc[j][nt][3] = bias[nt][1];
        }
#pragma unroll 2
      for (int ks = 0; ks < d.nks; ++ks) {
        const int2 kt = ktab[2 * ks + akh];
        uint32_t a[2][4];
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          uint32_t off = (uint32_t)((pbase[j] + kt.x) * cb + kt.y);
          off ^= ((off >> 7) & smask) << 4;   // the TMA swizzle of 32 / 64 / 128-byte rows
          ldsm4(fbase + off, a[j]);
        }
        if constexpr (NTU == 1) {   // one n-tile (K = 8): its two k halves only
          uint32_t b0, b1;
          asm volatile("ldmatrix.sync.aligned.m8n8.x2.shared.b16 {%0, %1}, [%2];"
                       : "=r"(b0), "=r"(b1)
                       : "r"(wbase + (uint32_t)(ks * 2 * d.Kp * 16) + boff_lane));
#pragma unroll
          for (int j = 0; j < 2; ++j) mma16816(acc[j][0], a[j], b0, b1);
        } else {
#pragma unroll
          for (int np = 0; np < NT2; ++np) {
            uint32_t bb[4];
            ldsm4(wbase + (uint32_t)((ks * 2 * d.Kp + np * 16) * 16) + boff_lane, bb);
#pragma unroll
            for (int j = 0; j < 2; ++j) {
              mma16816(acc[j][2 * np], a[j], bb[0], bb[1]);
              mma16816(acc[j][2 * np + 1], a[j], bb[2], bb[3]);
            }
          }
        }
      }
#pragma unroll
      for (int j = 0; j < 2; ++j)
#pragma unroll
        for (int hf = 0; hf < 2; ++hf) {
          const int q = (mt0 + j) * 16 + g + 8 * hf;
          if (q >= npx) continue;
          const int pn = fdiv(q, d.mpx, d.spx), rem = q - pn * pxt, py = fdiv(rem, d.mtw, d.stw), px = rem - py * d.TW;
          const int on = n0 + pn, oh = oh0 + py, ow = ow0 + px;
          if (on >= d.N || oh >= d.Ho || ow >= d.Wo) continue;
          __nv_bfloat16* yp = y + (((int64_t)on * d.Ho + oh) * d.Wo + ow) * d.K + 2 * t4;
#pragma unroll
          for (int nt = 0; nt < NTU; ++nt)
            if (nt * 8 < d.K)
              *reinterpret_cast<uint32_t*>(yp + nt * 8) = pk2(acc[j][nt][2 * hf], acc[j][nt][2 * hf + 1]);
        }
    }
    warp_arrive(&empty[b]);   // this warp is done with buffer b
  }
}

template <int NT2, int NTU>
void launch_t(const TileConvDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  static bool configured = false;
  static int sms = 148;
  if (!configured) {
    cudaFuncSetAttribute(tile_conv_kernel<NT2, NTU>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    configured = true;
  }
  int per_sm = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, tile_conv_kernel<NT2, NTU>, kTcThreads, d.smem_bytes);
  const int grid = std::min(d.ntiles, sms * std::max(per_sm, 1));
  launch_pdl(tile_conv_kernel<NT2, NTU>, dim3((unsigned)grid), dim3(kTcThreads), (size_t)d.smem_bytes, s, d, p, tcw);
}

}  // namespace

void launch_tile_conv(const TileConvDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  if (d.K == 8) return launch_t<1, 1>(d, tcw, p, s);
  switch (d.Kp / 16) {
    case 1: launch_t<1, 2>(d, tcw, p, s); break;
    case 2: launch_t<2, 4>(d, tcw, p, s); break;
    case 3: launch_t<3, 6>(d, tcw, p, s); break;
    default: launch_t<4, 8>(d, tcw, p, s); break;
  }
}

}  // namespace temco
