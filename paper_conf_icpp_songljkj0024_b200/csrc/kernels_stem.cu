// Small-Cin direct convolution on tensor cores (bf16 mode): the Tucker stem core
// on the 3-channel image (7x7 s2 for ResNet-50 / DenseNet-121, 3x3 s1 for the
// CIFAR ResNet-18) and VGG's first CP factor (1x1, 3 -> 8).
//
// A full-rank image mode is not decomposed (R17), so this conv reads the raw
// image: K = kh*kw*Cin is tiny (<= ~200) and the output has 8..64 channels.
// It is HBM-bound (AI ~ 10-20 flop/B), so the design goal is to read the image
// once with no im2col materialisation:
//   * a CTA stages the input footprint of a 16 x 32 output tile in SMEM as bf16,
//     pixel stride Cp = Cin rounded up to even (zero channel padding), so each
//     kernel row (kw pixels x Cp channels) is a contiguous run of SMEM;
//   * the implicit-GEMM A fragments of mma.sync.m16n8k16 (row = output pixel,
//     column = (kernel row, pixel-in-row, channel)) are single 32-bit LDS from
//     that footprint (pairs never straddle a kernel row because Cp is even);
//     K is padded to k-steps of 16 with zero weights;
//   * the B fragments (weights, bf16) are register-resident for the whole CTA;
//   * fp32 accumulation, bf16 NHWC output written straight from the fragments
//     (four lanes cover one pixel's 16-byte channel group: coalesced rows).
#include <cuda_bf16.h>

#include <algorithm>

#include "kernels.h"

namespace temco {

namespace {

// output tile (rows x cols): 16 x 32 (8 warps x 4 m-tiles of 16 pixels); strided stems whose
// 16 x 32 footprint overflows the stage (AlexNet's 11x11 / s4) take 8 x 16 (one m-tile per warp)
constexpr int kStTH = 16, kStTW = 32;
constexpr int kStThreads = 256;

constexpr int kStCPT = 6;   // footprint chunks (16 B of an image row) per thread and tile

struct StemGeo {
  int TH, TW, MPW;        // output tile, m-tiles (16 pixels) per warp
  int Cp, rowK, KS, NT;   // padded channels, elements per kernel row, k-steps, n-tiles
  int PR, PC, rowlen;     // footprint rows / pixels, elements per footprint row
  int ncr;                // 16-byte image-row chunks covering one footprint row
  int cmagic;             // (j * cmagic) >> 17 == j / Cin for j < 2048
  int buf;                // 32-bit words of one footprint buffer (incl. slack)
  int smem;               // bytes (two buffers)
};

StemGeo stem_geo(const ConvDesc& d, int TH = kStTH, int TW = kStTW) {
  StemGeo g;
  g.TH = TH;
  g.TW = TW;
  g.MPW = TH * TW / 16 / 8;
  g.Cp = (d.C + 1) / 2 * 2;
  g.rowK = d.kw * g.Cp;
  g.KS = (d.kh * g.rowK + 15) / 16;
  g.NT = d.K / 8;
  g.PR = (TH - 1) * d.sh + d.kh;
  g.PC = (TW - 1) * d.sw + d.kw;
  g.rowlen = g.PC * g.Cp;
  g.ncr = (g.PC * d.C + 7) / 8 + 1;
  g.cmagic = ((1 << 17) + d.C - 1) / d.C;
  // + slack: padded k columns past the last kernel row read (finite) footprint data
  g.buf = (g.PR * g.rowlen + 64) / 2;
  // + SMEM B fragments and k-offsets (long K)
  g.smem = g.buf * 4 * 2 + (g.KS > 16 ? g.KS * g.NT * 32 * 8 + g.KS * 8 * 4 : 0);
  return g;
}

__device__ __forceinline__ void mma_bf16_16816(float* c, const uint32_t* a, uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
  __nv_bfloat162 h = __floats2bfloat162_rn(lo, hi);
  return *reinterpret_cast<uint32_t*>(&h);
}

template <int KS, int NT>
__global__ void __launch_bounds__(kStThreads, 2) conv_stem_kernel(ConvDesc d, StemGeo g, RunPtrs p, int tiles_w,
                                                               int tiles_h) {
  extern __shared__ __align__(16) __nv_bfloat16 xs[];   // two footprint buffers of g.buf elements
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int gq = lane >> 2, tq = lane & 3;
  // ---- per-thread k-pair offsets into a pixel's footprint window and the B fragments
  const float* wf = p.params + d.w;   // fp32 [K][kh][kw][Cin]
  // long K (AlexNet's 11x11 stem, 31 k-steps): the B fragments live in SMEM (one LDS.64 per
  // k-step) instead of 62 registers per n-tile
  constexpr bool kBs = KS > 16;
  uint2* bs = reinterpret_cast<uint2*>(reinterpret_cast<uint32_t*>(xs) + 2 * g.buf);
  int* os = reinterpret_cast<int*>(bs + KS * NT * 32);   // [ks][h][tq]
  int off[kBs ? 1 : KS][2];
  uint32_t bfr[kBs ? 1 : NT][kBs ? 1 : KS][2];
#pragma unroll
  for (int ks = 0; ks < KS; ++ks)
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int k = ks * 16 + 2 * tq + 8 * h;           // even: the pair (k, k+1) shares its kernel row
      const int kr = k / g.rowK, j = k - kr * g.rowK;
      if constexpr (kBs) {
        if (gq == 0) os[(ks * 2 + h) * 4 + tq] = kr < d.kh ? 2 * (kr * g.rowlen + j) : 0;   // bytes
      } else {
        off[ks][h] = kr < d.kh ? 2 * (kr * g.rowlen + j) : 0;   // bytes (even element offsets)
      }
#pragma unroll
      for (int nt = 0; nt < NT; ++nt) {
        const int o = nt * 8 + gq;
        float w2[2];
#pragma unroll
        for (int e = 0; e < 2; ++e) {
          const int jj = j + e, px = jj / g.Cp, c = jj - px * g.Cp;
          w2[e] = (kr < d.kh && c < d.C) ? wf[(((int64_t)o * d.kh + kr) * d.kw + px) * d.C + c] : 0.f;
        }
        if constexpr (kBs)
          reinterpret_cast<uint32_t*>(&bs[(ks * NT + nt) * 32 + lane])[h] = pack2(w2[0], w2[1]);
        else
          bfr[nt][ks][h] = pack2(w2[0], w2[1]);
      }
    }
  float bias[NT][2];
#pragma unroll
  for (int nt = 0; nt < NT; ++nt)
#pragma unroll
    for (int e = 0; e < 2; ++e) bias[nt][e] = d.b >= 0 ? p.params[d.b + nt * 8 + 2 * tq + e] : 0.f;
  // both buffers start zeroed: the pad channels and the slack are never written again
  // (2 buffers x g.buf words); the barrier orders the zeroing before the first footprint
  // store (compute-sanitizer racecheck: the stores of store() overlapped the zeroing)
  for (int i = threadIdx.x; i < 2 * g.buf; i += kStThreads) reinterpret_cast<uint32_t*>(xs)[i] = 0u;
  __syncthreads();
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(const_cast<void*>(loc_ptr(d.y, p)));
  const uint4* x4 = reinterpret_cast<const uint4*>(loc_ptr(d.x, p));
  const int rowC = d.W * d.C;            // image row in elements (% 8 == 0)
  const int fl = g.PC * d.C;             // footprint row in elements
  const int ntiles = d.N * tiles_w * tiles_h;
  // footprint of a tile as 16-byte chunks of image rows, kStCPT chunks per thread in registers
  uint4 v[kStCPT];
  auto load_any = [&](int tile) {
    const int n = tile / (tiles_w * tiles_h);
    const int h0 = (tile / tiles_w) % tiles_h * g.TH, w0 = tile % tiles_w * g.TW;
    const int hi0 = h0 * d.sh - d.ph, e0 = (w0 * d.sw - d.pw) * d.C;
    const int a0 = e0 >= 0 ? e0 / 8 : -((7 - e0) / 8);
#pragma unroll
    for (int q = 0; q < kStCPT; ++q) {
      const int i = threadIdx.x + q * kStThreads;
      const int r = i / g.ncr, ch = a0 + (i - r * g.ncr);
      const int hi = hi0 + r;
      const bool ok = i < g.PR * g.ncr && hi >= 0 && hi < d.H && ch >= 0 && ch * 8 < rowC;
      v[q] = ok ? __ldg(x4 + (((int64_t)n * d.H + hi) * rowC) / 8 + ch) : make_uint4(0, 0, 0, 0);
    }
  };
  auto store_any = [&](int tile, __nv_bfloat16* buf) {
    const int w0 = tile % tiles_w * g.TW;
    const int e0 = (w0 * d.sw - d.pw) * d.C;
    const int a0 = e0 >= 0 ? e0 / 8 : -((7 - e0) / 8);
#pragma unroll
    for (int q = 0; q < kStCPT; ++q) {
      const int i = threadIdx.x + q * kStThreads;
      if (i >= g.PR * g.ncr) break;
      const int r = i / g.ncr;
      const int j0 = (a0 + (i - r * g.ncr)) * 8 - e0;   // footprint-row position of the chunk's element 0
      const uint32_t w[4] = {v[q].x, v[q].y, v[q].z, v[q].w};
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        const int j = j0 + e;
        if (j >= 0 && j < fl) {
          const int px = (j * g.cmagic) >> 17, c = j - px * d.C;
          reinterpret_cast<unsigned short*>(buf)[r * g.rowlen + px * g.Cp + c] =
              (unsigned short)(w[e >> 1] >> ((e & 1) * 16));
        }
      }
    }
  };
  // 3-channel images (every stem here): 8-pixel groups -- 3 chunks of 16 bytes = 24 elements = 8 whole
  // pixels -- so each pixel goes to SMEM as one 8-byte (c0, c1, c2, 0) store with compile-time element
  // extraction, instead of 8 scalar stores per chunk with per-element index arithmetic
  const bool g3 = d.C == 3 && g.Cp == 4;
  auto grp = [&](int tile, int& gA, int& ng, int& fx0) {
    const int w0 = tile % tiles_w * g.TW;
    fx0 = w0 * d.sw - d.pw;
    gA = fx0 >= 0 ? fx0 / 8 : -((7 - fx0) / 8);
    const int e = fx0 + g.PC;   // one past the last footprint column
    ng = (e >= 0 ? (e + 7) / 8 : -((-e) / 8)) - gA;
  };
  auto load3 = [&](int tile) {
    const int n = tile / (tiles_w * tiles_h);
    const int h0 = (tile / tiles_w) % tiles_h * g.TH;
    const int hi0 = h0 * d.sh - d.ph;
    int gA, ng, fx0;
    grp(tile, gA, ng, fx0);
#pragma unroll
    for (int q = 0; q < kStCPT / 3; ++q) {
      const int i = threadIdx.x + q * kStThreads;
      const int r = i / ng, gg = i - r * ng, hi = hi0 + r;
      const bool rok = i < g.PR * ng && hi >= 0 && hi < d.H;
      const int64_t rowb = (((int64_t)n * d.H + hi) * rowC) / 8;
#pragma unroll
      for (int c3 = 0; c3 < 3; ++c3) {
        const int ch = (gA + gg) * 3 + c3;
        v[q * 3 + c3] = (rok && ch >= 0 && ch * 8 < rowC) ? __ldg(x4 + rowb + ch) : make_uint4(0, 0, 0, 0);
      }
    }
  };
  auto store3 = [&](int tile, __nv_bfloat16* buf) {
    int gA, ng, fx0;
    grp(tile, gA, ng, fx0);
#pragma unroll
    for (int q = 0; q < kStCPT / 3; ++q) {
      const int i = threadIdx.x + q * kStThreads;
      if (i >= g.PR * ng) break;
      const int r = i / ng, gg = i - r * ng;
      const uint32_t w[12] = {v[3 * q].x, v[3 * q].y, v[3 * q].z, v[3 * q].w, v[3 * q + 1].x, v[3 * q + 1].y,
                              v[3 * q + 1].z, v[3 * q + 1].w, v[3 * q + 2].x, v[3 * q + 2].y, v[3 * q + 2].z,
                              v[3 * q + 2].w};
      const int fc0 = (gA + gg) * 8 - fx0;
#pragma unroll
      for (int pp = 0; pp < 8; ++pp) {
        const int fc = fc0 + pp;
        if (fc < 0 || fc >= g.PC) continue;
        const int e = 3 * pp;   // compile-time element positions of this pixel's three channels
        const uint32_t c0 = (w[e >> 1] >> ((e & 1) * 16)) & 0xFFFFu;
        const uint32_t c1 = (w[(e + 1) >> 1] >> (((e + 1) & 1) * 16)) & 0xFFFFu;
        const uint32_t c2 = (w[(e + 2) >> 1] >> (((e + 2) & 1) * 16)) & 0xFFFFu;
        *reinterpret_cast<uint2*>(reinterpret_cast<unsigned short*>(buf) + r * g.rowlen + fc * 4) =
            make_uint2(c0 | (c1 << 16), c2);
      }
    }
  };
  auto load = [&](int tile) {
    if (g3) load3(tile);
    else load_any(tile);
  };
  auto store = [&](int tile, __nv_bfloat16* buf) {
    if (g3) store3(tile, buf);
    else store_any(tile, buf);
  };
  int tile = blockIdx.x;
  pdl_wait();
  pdl_trigger_early();
  if (tile < ntiles) load(tile);
  int b = 0;
  for (; tile < ntiles; tile += gridDim.x, b ^= 1) {
    __nv_bfloat16* buf = xs + b * g.buf * 2;
    store(tile, buf);
    __syncthreads();
    const int n = tile / (tiles_w * tiles_h);
    const int h0 = (tile / tiles_w) % tiles_h * g.TH, w0 = tile % tiles_w * g.TW;
    if (tile + (int)gridDim.x < ntiles) load(tile + gridDim.x);   // in flight during the MMAs
    // ---- MPW m-tiles per warp: m-tile gm covers output row gm / (TW / 16), 16 columns
#pragma unroll 1
    for (int gm = warp * g.MPW; gm < (warp + 1) * g.MPW; ++gm) {
      // m-tile gm: output row gm / (TW / 16), columns 16 (gm % (TW / 16)) .. (TW is 16 or 32)
      const int orow = g.TW == 32 ? gm >> 1 : gm, ocol = g.TW == 32 ? (gm & 1) * 16 : 0;
      // byte addresses of the fragment rows gq, gq + 8 (element offsets are even: 4-byte aligned words)
      const uint8_t* xb0 = reinterpret_cast<const uint8_t*>(buf) + 2 * ((orow * d.sh) * g.rowlen + ((ocol + gq) * d.sw) * g.Cp);
      const uint8_t* xb1 = xb0 + 2 * 8 * d.sw * g.Cp;
      float acc[NT][4];
#pragma unroll
      for (int nt = 0; nt < NT; ++nt) {
        acc[nt][0] = acc[nt][2] = bias[nt][0];
        acc[nt][1] = acc[nt][3] = bias[nt][1];
      }
#pragma unroll
      for (int ks = 0; ks < KS; ++ks) {
        uint32_t a[4];
        int o0, o1;
        if constexpr (kBs) {
          o0 = os[ks * 8 + tq];
          o1 = os[ks * 8 + 4 + tq];
        } else {
          o0 = off[ks][0];
          o1 = off[ks][1];
        }
        a[0] = *reinterpret_cast<const uint32_t*>(xb0 + o0);
        a[1] = *reinterpret_cast<const uint32_t*>(xb1 + o0);
        a[2] = *reinterpret_cast<const uint32_t*>(xb0 + o1);
        a[3] = *reinterpret_cast<const uint32_t*>(xb1 + o1);
#pragma unroll
        for (int nt = 0; nt < NT; ++nt) {
          if constexpr (kBs) {
            const uint2 bb = bs[(ks * NT + nt) * 32 + lane];
            mma_bf16_16816(acc[nt], a, bb.x, bb.y);
          } else {
            mma_bf16_16816(acc[nt], a, bfr[nt][ks][0], bfr[nt][ks][1]);
          }
        }
      }
      const int oy = h0 + orow;
      if (oy >= d.Ho) continue;
#pragma unroll
      for (int hf = 0; hf < 2; ++hf) {
        const int ox = w0 + ocol + gq + 8 * hf;
        if (ox >= d.Wo) continue;
        __nv_bfloat16* yp = y + (((int64_t)n * d.Ho + oy) * d.Wo + ox) * d.K + 2 * tq;
#pragma unroll
        for (int nt = 0; nt < NT; ++nt)
          *reinterpret_cast<uint32_t*>(yp + nt * 8) = pack2(acc[nt][2 * hf], acc[nt][2 * hf + 1]);
      }
    }
  }
}

template <int KS, int NT>
void launch_stem_t(const ConvDesc& d, const StemGeo& g, const RunPtrs& p, cudaStream_t s) {
  static bool configured = false;
  static int sms = 148;
  if (!configured) {
    cudaFuncSetAttribute(conv_stem_kernel<KS, NT>, cudaFuncAttributeMaxDynamicSharedMemorySize, 96 * 1024);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    configured = true;
  }
  int per_sm = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, conv_stem_kernel<KS, NT>, kStThreads, g.smem);
  const int tw = (d.Wo + g.TW - 1) / g.TW, th = (d.Ho + g.TH - 1) / g.TH;
  const int ntiles = d.N * tw * th;
  const int grid = std::min(ntiles, sms * std::max(per_sm, 1));
  launch_pdl(conv_stem_kernel<KS, NT>, dim3((unsigned)grid), dim3(kStThreads), g.smem, s, d, g, p, tw, th);
}

// 1x1 stride-1 conv on the image (VGG's first CP factor, 3 -> 8): a pure per-pixel
// map, HBM-bound on the 6-byte pixel read + 16-byte write -- one thread per pixel,
// weights in registers, fp32 FMAs, one 16-byte store
template <int CIN>
__global__ void __launch_bounds__(256) conv_pw_small_kernel(ConvDesc d, RunPtrs p) {
  float w[8][CIN], b[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) {
#pragma unroll
    for (int c = 0; c < CIN; ++c) w[k][c] = p.params[d.w + k * CIN + c];
    b[k] = d.b >= 0 ? p.params[d.b + k] : 0.f;
  }
  pdl_wait();
  pdl_trigger_early();
  const unsigned short* x = reinterpret_cast<const unsigned short*>(loc_ptr(d.x, p));
  uint4* y = reinterpret_cast<uint4*>(const_cast<void*>(loc_ptr(d.y, p)));
  const int64_t npix = (int64_t)d.N * d.H * d.W;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < npix; i += (int64_t)gridDim.x * blockDim.x) {
    float xv[CIN];
#pragma unroll
    for (int c = 0; c < CIN; ++c) xv[c] = __uint_as_float((uint32_t)__ldg(x + i * CIN + c) << 16);
    float o[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      o[k] = b[k];
#pragma unroll
      for (int c = 0; c < CIN; ++c) o[k] = fmaf(w[k][c], xv[c], o[k]);
    }
    y[i] = make_uint4(pack2(o[0], o[1]), pack2(o[2], o[3]), pack2(o[4], o[5]), pack2(o[6], o[7]));
  }
}

bool stem_fits(const ConvDesc& d, const StemGeo& g) {
  const bool g3_fits = d.C != 3 || g.PR * ((g.PC + 7) / 8 + 1) <= kStCPT / 3 * kStThreads;   // 8-pixel groups
  return g.smem <= 96 * 1024 && g.PR * g.ncr <= kStCPT * kStThreads && g.PC * d.C < 2048 && g3_fits;
}

StemGeo stem_pick(const ConvDesc& d) {
  const StemGeo g = stem_geo(d);
  return stem_fits(d, g) ? g : stem_geo(d, 8, 16);
}

}  // namespace

bool conv_stem_ok(const ConvDesc& d) {
  if (d.x.dtype != DT_BF16 || d.y.dtype != DT_BF16 || d.groups != 1 || d.C > 8 || d.K % 8 || d.sh != d.sw) return false;
  const StemGeo g = stem_pick(d);
  const bool shape = (g.NT == 1 || g.NT == 2) && (g.KS == 1 || g.KS == 3 || g.KS == 13 || g.KS == 31);
  return shape && stem_fits(d, g) && (d.W * d.C) % 8 == 0;
}

void launch_conv_stem(const ConvDesc& d, const RunPtrs& p, cudaStream_t s) {
  if (d.kh == 1 && d.kw == 1 && d.sh == 1 && d.ph == 0 && d.pw == 0 && d.C == 3 && d.K == 8) {
    const int64_t npix = (int64_t)d.N * d.H * d.W;
    const int grid = (int)std::min<int64_t>((npix + 255) / 256, 148LL * 16);
    launch_pdl(conv_pw_small_kernel<3>, dim3(grid), dim3(256), 0, s, d, p);
    return;
  }
  const StemGeo g = stem_pick(d);
#define TEMCO_STEM_CASE(ks, nt) \
  if (g.KS == ks && g.NT == nt) return launch_stem_t<ks, nt>(d, g, p, s);
  TEMCO_STEM_CASE(1, 1)
  TEMCO_STEM_CASE(3, 1)
  TEMCO_STEM_CASE(13, 1)
  TEMCO_STEM_CASE(1, 2)
  TEMCO_STEM_CASE(3, 2)
  TEMCO_STEM_CASE(13, 2)
  TEMCO_STEM_CASE(31, 1)
#undef TEMCO_STEM_CASE
}

}  // namespace temco
