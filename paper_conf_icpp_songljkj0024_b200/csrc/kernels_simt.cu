// Generic SIMT kernels (fp32 arithmetic on fp32 / bf16 NHWC storage).
//
// These cover every step shape the planner can emit and are the fp32-mode
// path (no TF32: reading R22, the 1e-4 parity bar).  The tcgen05 kernels in
// kernels_tc.cu replace the hot fused groups in bf16 mode.
#include <cuda_bf16.h>

#include <algorithm>
#include <cfloat>
#include <cstdint>
#include <cstdlib>

#include "kernels.h"

namespace temco {

namespace {

__device__ __forceinline__ float ldv(const void* base, int64_t i, int dt) {
  return dt == DT_BF16 ? __bfloat162float(reinterpret_cast<const __nv_bfloat16*>(base)[i])
                       : reinterpret_cast<const float*>(base)[i];
}

__device__ __forceinline__ void stv(void* base, int64_t i, float v, int dt) {
  if (dt == DT_BF16)
    reinterpret_cast<__nv_bfloat16*>(base)[i] = __float2bfloat16_rn(v);
  else
    reinterpret_cast<float*>(base)[i] = v;
}

inline int grid_for(int64_t total, int block) {
  int64_t g = (total + block - 1) / block;
  const int64_t cap = 148LL * 32;
  return (int)(g < cap ? (g > 0 ? g : 1) : cap);
}

// ---------------------------------------------------------------------------
// small-Cin direct convolution (the stem core on the 3-channel image, CP first
// factors on it): a 16 x 32 output tile per CTA, its input footprint staged in
// SMEM as fp32, each thread two output rows x 8 output channels (weights are
// warp-broadcast SMEM reads shared by the two pixels).  gridDim.z = K / 8.
// ---------------------------------------------------------------------------
constexpr int kSmTH = 16, kSmTW = 32, kSmKC = 8;

__global__ void __launch_bounds__(256) conv_small_kernel(ConvDesc d, RunPtrs p, int tiles_w, int tiles_h) {
  extern __shared__ float sm[];
  const int Cin = d.C;
  const int ir = (kSmTH - 1) * d.sh + d.kh, ic = (kSmTW - 1) * d.sw + d.kw;
  const int taps = d.kh * d.kw;
  float* xs = sm;                                   // [ir][ic][Cin]
  float* ws = sm + (ir * ic * Cin + 3) / 4 * 4;     // [tap][c][8], 16-byte aligned
  const int tile = blockIdx.x;
  const int n = tile / (tiles_w * tiles_h);
  const int h0 = (tile / tiles_w) % tiles_h * kSmTH, w0 = tile % tiles_w * kSmTW;
  const int k0 = blockIdx.y * kSmKC;
  const void* x = loc_ptr(d.x, p);
  // stage the input footprint (zero padding outside the image)
  const int hi0 = h0 * d.sh - d.ph, wi0 = w0 * d.sw - d.pw;
  const int rowlen = ic * Cin;
  for (int i = threadIdx.x; i < ir * rowlen; i += blockDim.x) {
    const int r = i / rowlen, e = i % rowlen;
    const int hi = hi0 + r, wi = wi0 + e / Cin, c = e % Cin;
    float v = 0.f;
    if (hi >= 0 && hi < d.H && wi >= 0 && wi < d.W)
      v = ldv(x, (((int64_t)n * d.H + hi) * d.W + wi) * Cin + c, d.x.dtype);
    xs[i] = v;
  }
  for (int i = threadIdx.x; i < taps * Cin * kSmKC; i += blockDim.x) {
    const int j = i % kSmKC, tc = i / kSmKC;
    const int k = k0 + j;
    ws[i] = k < d.K ? p.params[d.w + (int64_t)k * taps * Cin + tc] : 0.f;
  }
  __syncthreads();
  const int tx = threadIdx.x % kSmTW, ty = threadIdx.x / kSmTW;   // rows ty and ty + 8
  float acc0[kSmKC], acc1[kSmKC];
#pragma unroll
  for (int j = 0; j < kSmKC; ++j) {
    const float b = (d.b >= 0 && k0 + j < d.K) ? p.params[d.b + k0 + j] : 0.f;
    acc0[j] = b;
    acc1[j] = b;
  }
  const int r8 = 8 * d.sh * rowlen;
  for (int a = 0; a < d.kh; ++a)
    for (int bb = 0; bb < d.kw; ++bb) {
      const float* xp = xs + (ty * d.sh + a) * rowlen + (tx * d.sw + bb) * Cin;
      const float* wp = ws + (a * d.kw + bb) * Cin * kSmKC;
      for (int c = 0; c < Cin; ++c) {
        const float x0 = xp[c], x1 = xp[r8 + c];
        const float4 wa = reinterpret_cast<const float4*>(wp + c * kSmKC)[0];
        const float4 wb = reinterpret_cast<const float4*>(wp + c * kSmKC)[1];
        const float w8[8] = {wa.x, wa.y, wa.z, wa.w, wb.x, wb.y, wb.z, wb.w};
#pragma unroll
        for (int j = 0; j < kSmKC; ++j) {
          acc0[j] = fmaf(w8[j], x0, acc0[j]);
          acc1[j] = fmaf(w8[j], x1, acc1[j]);
        }
      }
    }
  void* y = const_cast<void*>(loc_ptr(d.y, p));
  const int wo = w0 + tx;
#pragma unroll
  for (int s = 0; s < 2; ++s) {
    const int ho = h0 + ty + 8 * s;
    if (ho >= d.Ho || wo >= d.Wo) continue;
    const float* acc = s ? acc1 : acc0;
    const int64_t base = (((int64_t)n * d.Ho + ho) * d.Wo + wo) * d.K + k0;
    if (d.y.dtype == DT_BF16 && k0 + kSmKC <= d.K && d.K % 8 == 0) {
      uint4 pk;
      __nv_bfloat162 h01 = __floats2bfloat162_rn(acc[0], acc[1]), h23 = __floats2bfloat162_rn(acc[2], acc[3]);
      __nv_bfloat162 h45 = __floats2bfloat162_rn(acc[4], acc[5]), h67 = __floats2bfloat162_rn(acc[6], acc[7]);
      pk.x = *reinterpret_cast<uint32_t*>(&h01);
      pk.y = *reinterpret_cast<uint32_t*>(&h23);
      pk.z = *reinterpret_cast<uint32_t*>(&h45);
      pk.w = *reinterpret_cast<uint32_t*>(&h67);
      *reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(y) + base) = pk;
    } else {
      for (int j = 0; j < kSmKC && k0 + j < d.K; ++j) stv(y, base + j, acc[j], d.y.dtype);
    }
  }
}

int conv_small_smem(const ConvDesc& d) {
  const int ir = (kSmTH - 1) * d.sh + d.kh, ic = (kSmTW - 1) * d.sw + d.kw;
  return ((ir * ic * d.C + 3) / 4 * 4 + d.kh * d.kw * d.C * kSmKC) * 4;
}

// ---------------------------------------------------------------------------
// reduced-rank core convolution (Tucker core K x K on R_in -> R_out channels,
// the 1x1 cores, CP pointwise factors): memory-bound work (AI < 150 flop/B at
// R <= 64), so a direct SIMT kernel with coalesced 16-byte staging beats an
// implicit GEMM whose tiles are dominated by tensor-core issue latency.
// CTA: a box of ni images x th rows x tw columns of output pixels (one pixel
// per thread), kc output channels (gridDim.y = K / kc).  The input footprint
// is staged in SMEM as bf16 (16-byte row segments), the weights as fp32
// [tap][cin][kc] (warp-broadcast float4 reads); fp32 accumulation.
// ---------------------------------------------------------------------------
struct RankTile {
  int ni, th, tw, kc, fr, fc;   // images, rows, cols per tile; output channels per CTA; footprint rows / cols
  int tiles_w, tiles_h, tiles_n;
  int smem;
};

__host__ __device__ inline RankTile rank_tile(const ConvDesc& d) {
  RankTile t;
  t.tw = d.Wo <= 32 ? d.Wo : (d.Wo + (d.Wo + 31) / 32 - 1) / ((d.Wo + 31) / 32);
  t.th = 256 / t.tw < d.Ho ? 256 / t.tw : d.Ho;
  t.ni = (t.th == d.Ho) ? (256 / (t.tw * t.th) < d.N ? 256 / (t.tw * t.th) : d.N) : 1;
  if (t.ni < 1) t.ni = 1;
  t.kc = d.K <= 16 ? d.K : 16;
  t.fr = (t.th - 1) * d.sh + d.kh;
  t.fc = (t.tw - 1) * d.sw + d.kw;
  t.tiles_w = (d.Wo + t.tw - 1) / t.tw;
  t.tiles_h = (d.Ho + t.th - 1) / t.th;
  t.tiles_n = (d.N + t.ni - 1) / t.ni;
  t.smem = t.ni * t.fr * t.fc * d.C * 2 + d.kh * d.kw * d.C * t.kc * 4;
  return t;
}

template <int KC>
__global__ void __launch_bounds__(256) conv_rank_kernel(ConvDesc d, RankTile t, RunPtrs p) {
  pdl_wait();
  pdl_trigger_early();
  extern __shared__ __align__(16) unsigned char smr[];
  const int Cin = d.C;
  const int taps = d.kh * d.kw;
  float* ws = reinterpret_cast<float*>(smr);                                   // [tap][cin][KC]
  __nv_bfloat16* xs = reinterpret_cast<__nv_bfloat16*>(smr + taps * Cin * KC * 4);   // [img][fr][fc][cin]
  const int tile = blockIdx.x;
  const int tw_i = tile % t.tiles_w, th_i = (tile / t.tiles_w) % t.tiles_h, tn_i = tile / (t.tiles_w * t.tiles_h);
  const int n0 = tn_i * t.ni, h0 = th_i * t.th, w0 = tw_i * t.tw;
  const int k0 = blockIdx.y * KC;
  // weights [k][tap][cin] (params) -> [tap][cin][k] (SMEM, fp32)
  for (int i = threadIdx.x; i < taps * Cin * KC; i += blockDim.x) {
    const int k = i % KC, tc = i / KC;
    ws[i] = p.params[d.w + (int64_t)(k0 + k) * taps * Cin + tc];
  }
  // input footprint, 16-byte vectors (Cin % 8 == 0), zero padding
  const __nv_bfloat16* x = reinterpret_cast<const __nv_bfloat16*>(loc_ptr(d.x, p));
  const int hi0 = h0 * d.sh - d.ph, wi0 = w0 * d.sw - d.pw;
  const int cv = Cin / 8;
  const int nvec = t.ni * t.fr * t.fc * cv;
  for (int i = threadIdx.x; i < nvec; i += blockDim.x) {
    const int c8 = i % cv, pix = i / cv;
    const int col = pix % t.fc, row = (pix / t.fc) % t.fr, img = pix / (t.fc * t.fr);
    const int n = n0 + img, hi = hi0 + row, wi = wi0 + col;
    uint4 v = make_uint4(0, 0, 0, 0);
    if (n < d.N && hi >= 0 && hi < d.H && wi >= 0 && wi < d.W)
      v = __ldg(reinterpret_cast<const uint4*>(x + (((int64_t)n * d.H + hi) * d.W + wi) * Cin) + c8);
    reinterpret_cast<uint4*>(xs)[i] = v;
  }
  __syncthreads();
  const int px = threadIdx.x;
  const int img = px / (t.th * t.tw), r = (px / t.tw) % t.th, c = px % t.tw;
  const int n = n0 + img, ho = h0 + r, wo = w0 + c;
  if (img >= t.ni || n >= d.N || ho >= d.Ho || wo >= d.Wo) return;
  float acc[KC];
#pragma unroll
  for (int k = 0; k < KC; ++k) acc[k] = d.b >= 0 ? p.params[d.b + k0 + k] : 0.f;
  const __nv_bfloat16* xi = xs + ((size_t)img * t.fr * t.fc) * Cin;
  for (int a = 0; a < d.kh; ++a)
    for (int bb = 0; bb < d.kw; ++bb) {
      const __nv_bfloat16* xp = xi + ((size_t)(r * d.sh + a) * t.fc + (c * d.sw + bb)) * Cin;
      const float* wp = ws + (a * d.kw + bb) * Cin * KC;
      for (int c8 = 0; c8 < cv; ++c8) {
        const uint4 u = reinterpret_cast<const uint4*>(xp)[c8];
        const uint32_t uw[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const float xv = __uint_as_float(j & 1 ? (uw[j / 2] & 0xFFFF0000u) : (uw[j / 2] << 16));
          const float4* w4 = reinterpret_cast<const float4*>(wp + (c8 * 8 + j) * KC);
#pragma unroll
          for (int k4 = 0; k4 < KC / 4; ++k4) {
            const float4 w = w4[k4];
            acc[4 * k4 + 0] = fmaf(xv, w.x, acc[4 * k4 + 0]);
            acc[4 * k4 + 1] = fmaf(xv, w.y, acc[4 * k4 + 1]);
            acc[4 * k4 + 2] = fmaf(xv, w.z, acc[4 * k4 + 2]);
            acc[4 * k4 + 3] = fmaf(xv, w.w, acc[4 * k4 + 3]);
          }
        }
      }
    }
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(const_cast<void*>(loc_ptr(d.y, p)));
  __nv_bfloat16* yp = y + (((int64_t)n * d.Ho + ho) * d.Wo + wo) * d.K + k0;
#pragma unroll
  for (int k8 = 0; k8 < KC / 8; ++k8) {
    uint4 pk;
    __nv_bfloat162 h0v = __floats2bfloat162_rn(acc[8 * k8 + 0], acc[8 * k8 + 1]);
    __nv_bfloat162 h1v = __floats2bfloat162_rn(acc[8 * k8 + 2], acc[8 * k8 + 3]);
    __nv_bfloat162 h2v = __floats2bfloat162_rn(acc[8 * k8 + 4], acc[8 * k8 + 5]);
    __nv_bfloat162 h3v = __floats2bfloat162_rn(acc[8 * k8 + 6], acc[8 * k8 + 7]);
    pk.x = *reinterpret_cast<uint32_t*>(&h0v);
    pk.y = *reinterpret_cast<uint32_t*>(&h1v);
    pk.z = *reinterpret_cast<uint32_t*>(&h2v);
    pk.w = *reinterpret_cast<uint32_t*>(&h3v);
    reinterpret_cast<uint4*>(yp)[k8] = pk;
  }
}

// ---------------------------------------------------------------------------
// depthwise (CP factor) convolution, bf16 NHWC: memory-bound, so one thread
// per (output pixel, 8-channel group) with 16-byte vector loads / stores --
// consecutive threads cover consecutive 16-byte chunks of a pixel row (fully
// coalesced), the kh x kw taps of neighbouring threads hit L1 / L2.
// ---------------------------------------------------------------------------
// vertical 3x1 CP factor (stride 1): a thread walks a strip of kColRows output
// rows of one (column, 8-channel group) with a sliding window -- the strip's
// kColRows + 2 input rows are loaded once, all in flight together
constexpr int kColRows = 8;
__global__ void __launch_bounds__(256) dwconv_col_kernel(ConvDesc d, RunPtrs p) {
  const __nv_bfloat16* x = reinterpret_cast<const __nv_bfloat16*>(loc_ptr(d.x, p));
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(const_cast<void*>(loc_ptr(d.y, p)));
  const int cg = d.C / 8;
  const int per_row = d.Wo * cg;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= per_row) return;
  const int wo = idx / cg, g = idx - wo * cg;
  const int spi = (d.Ho + kColRows - 1) / kColRows;     // strips per image
  float w[3][8], bias[8];
#pragma unroll
  for (int t = 0; t < 3; ++t) {
    const float4* w4 = reinterpret_cast<const float4*>(p.params + d.w2 + t * d.C + g * 8);
    const float4 wa = __ldg(w4), wb = __ldg(w4 + 1);
    w[t][0] = wa.x; w[t][1] = wa.y; w[t][2] = wa.z; w[t][3] = wa.w;
    w[t][4] = wb.x; w[t][5] = wb.y; w[t][6] = wb.z; w[t][7] = wb.w;
  }
#pragma unroll
  for (int j = 0; j < 8; ++j) bias[j] = d.b >= 0 ? __ldg(p.params + d.b + g * 8 + j) : 0.f;
  pdl_wait();
  pdl_trigger_early();
  for (int st = blockIdx.y; st < d.N * spi; st += gridDim.y) {
    const int n = st / spi, h0 = (st - n * spi) * kColRows;
    uint4 v[kColRows + 2];
#pragma unroll
    for (int r = 0; r < kColRows + 2; ++r) {
      const int hi = h0 - d.ph + r;
      v[r] = make_uint4(0, 0, 0, 0);
      if (hi >= 0 && hi < d.H && h0 + r - 2 < d.Ho)
        v[r] = __ldg(reinterpret_cast<const uint4*>(x + (((int64_t)n * d.H + hi) * d.W + wo) * d.C) + g);
    }
#pragma unroll
    for (int r = 0; r < kColRows; ++r) {
      if (h0 + r >= d.Ho) break;
      float acc[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) acc[j] = bias[j];
#pragma unroll
      for (int t = 0; t < 3; ++t) {
        const uint32_t uw[4] = {v[r + t].x, v[r + t].y, v[r + t].z, v[r + t].w};
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const float xv = __uint_as_float(j & 1 ? (uw[j / 2] & 0xFFFF0000u) : (uw[j / 2] << 16));
          acc[j] = fmaf(xv, w[t][j], acc[j]);
        }
      }
      uint4 pk;
      __nv_bfloat162 h0v = __floats2bfloat162_rn(acc[0], acc[1]), h1v = __floats2bfloat162_rn(acc[2], acc[3]);
      __nv_bfloat162 h2v = __floats2bfloat162_rn(acc[4], acc[5]), h3v = __floats2bfloat162_rn(acc[6], acc[7]);
      pk.x = *reinterpret_cast<uint32_t*>(&h0v);
      pk.y = *reinterpret_cast<uint32_t*>(&h1v);
      pk.z = *reinterpret_cast<uint32_t*>(&h2v);
      pk.w = *reinterpret_cast<uint32_t*>(&h3v);
      reinterpret_cast<uint4*>(y + (((int64_t)n * d.Ho + h0 + r) * d.Wo + wo) * d.C)[g] = pk;
    }
  }
}

// horizontal 1x3 CP factor (stride 1): one 16-byte load per thread; the left /
// right neighbours come from the lanes cg away (warp shuffles), only lanes whose
// neighbour lies outside the warp load it themselves
__global__ void __launch_bounds__(256) dwconv_row_kernel(ConvDesc d, RunPtrs p) {
  const __nv_bfloat16* x = reinterpret_cast<const __nv_bfloat16*>(loc_ptr(d.x, p));
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(const_cast<void*>(loc_ptr(d.y, p)));
  const int cg = d.C / 8;
  const int per_row = d.Wo * cg;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  const int lane = threadIdx.x & 31;
  const bool act = idx < per_row;
  const int wo = act ? idx / cg : 0, g = act ? idx - wo * cg : 0;
  float w[3][8], bias[8];
#pragma unroll
  for (int t = 0; t < 3; ++t) {
    const float4* w4 = reinterpret_cast<const float4*>(p.params + d.w2 + t * d.C + g * 8);
    const float4 wa = __ldg(w4), wb = __ldg(w4 + 1);
    w[t][0] = wa.x; w[t][1] = wa.y; w[t][2] = wa.z; w[t][3] = wa.w;
    w[t][4] = wb.x; w[t][5] = wb.y; w[t][6] = wb.z; w[t][7] = wb.w;
  }
#pragma unroll
  for (int j = 0; j < 8; ++j) bias[j] = d.b >= 0 ? __ldg(p.params + d.b + g * 8 + j) : 0.f;
  pdl_wait();
  pdl_trigger_early();
  constexpr int kRU = 4;   // rows per iteration: their loads in flight together
  const int rows = d.N * d.Ho;
  for (int row0 = blockIdx.y * kRU; row0 < rows; row0 += gridDim.y * kRU) {
  uint4 cr[kRU];
#pragma unroll
  for (int q = 0; q < kRU; ++q)
    cr[q] = (act && row0 + q < rows)
                ? __ldg(reinterpret_cast<const uint4*>(x + (int64_t)(row0 + q) * d.W * d.C) + g + (int64_t)wo * cg)
                : make_uint4(0, 0, 0, 0);
#pragma unroll
  for (int q = 0; q < kRU; ++q) {
    const int row = row0 + q;
    const uint4* xr = reinterpret_cast<const uint4*>(x + (int64_t)row * d.W * d.C) + g;   // Ho == H, stride 1
    const uint4 z = make_uint4(0, 0, 0, 0);
    const uint4 c = cr[q];
    uint4 v[3];
    v[1] = c;
#pragma unroll
    for (int side = 0; side < 2; ++side) {
      const int wi = wo - d.pw + 2 * side;      // left (side 0) / right (side 1) neighbour column
      uint4 s4;
      s4.x = side ? __shfl_down_sync(0xffffffffu, c.x, cg) : __shfl_up_sync(0xffffffffu, c.x, cg);
      s4.y = side ? __shfl_down_sync(0xffffffffu, c.y, cg) : __shfl_up_sync(0xffffffffu, c.y, cg);
      s4.z = side ? __shfl_down_sync(0xffffffffu, c.z, cg) : __shfl_up_sync(0xffffffffu, c.z, cg);
      s4.w = side ? __shfl_down_sync(0xffffffffu, c.w, cg) : __shfl_up_sync(0xffffffffu, c.w, cg);
      const bool inwarp = side ? lane + cg < 32 && idx + cg < per_row : lane >= cg;
      if (!(wi >= 0 && wi < d.W))
        s4 = z;
      else if (!inwarp && act && row < rows)
        s4 = __ldg(xr + (int64_t)wi * cg);
      v[2 * side] = s4;
    }
    if (!act || row >= rows) continue;
    float acc[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[j] = bias[j];
#pragma unroll
    for (int t = 0; t < 3; ++t) {
      const uint32_t uw[4] = {v[t].x, v[t].y, v[t].z, v[t].w};
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const float xv = __uint_as_float(j & 1 ? (uw[j / 2] & 0xFFFF0000u) : (uw[j / 2] << 16));
        acc[j] = fmaf(xv, w[t][j], acc[j]);
      }
    }
    uint4 pk;
    __nv_bfloat162 h0v = __floats2bfloat162_rn(acc[0], acc[1]), h1v = __floats2bfloat162_rn(acc[2], acc[3]);
    __nv_bfloat162 h2v = __floats2bfloat162_rn(acc[4], acc[5]), h3v = __floats2bfloat162_rn(acc[6], acc[7]);
    pk.x = *reinterpret_cast<uint32_t*>(&h0v);
    pk.y = *reinterpret_cast<uint32_t*>(&h1v);
    pk.z = *reinterpret_cast<uint32_t*>(&h2v);
    pk.w = *reinterpret_cast<uint32_t*>(&h3v);
    reinterpret_cast<uint4*>(y + ((int64_t)row * d.Wo + wo) * d.C)[g] = pk;
  }
  }
}

template <int KH, int KW>   // 0, 0: runtime kernel size (<= 9 taps)
__global__ void __launch_bounds__(256) dwconv_vec_kernel(ConvDesc d, RunPtrs p) {
  pdl_wait();
  pdl_trigger_early();
  // grid: x = chunks of (output column, 8-channel group) of one output row, y = output rows (n, ho):
  // 32-bit index math only (the 64-bit div/mod chain dominated the previous flat-index version)
  const __nv_bfloat16* x = reinterpret_cast<const __nv_bfloat16*>(loc_ptr(d.x, p));
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(const_cast<void*>(loc_ptr(d.y, p)));
  const int cg = d.C / 8;
  const int per_row = d.Wo * cg;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= per_row) return;
  const int wo = idx / cg, g = idx - wo * cg;
  for (int row = blockIdx.y; row < d.N * d.Ho; row += gridDim.y) {
    const int n = row / d.Ho, ho = row - n * d.Ho;
    // all taps' 16-byte loads in flight before any arithmetic (the CP factors are
    // 3x1 / 1x3: one load in flight per thread capped this kernel at ~2 TB/s)
    constexpr int kMaxTaps = KH > 0 ? KH * KW : 9;
    const int kw = KH > 0 ? KW : d.kw;
    uint4 v[kMaxTaps];
    const int taps = KH > 0 ? KH * KW : d.kh * d.kw;
#pragma unroll
    for (int t = 0; t < kMaxTaps; ++t) {
      v[t] = make_uint4(0, 0, 0, 0);
      if (t < taps) {
        const int a = t / kw, b = t - a * kw;
        const int hi = ho * d.sh - d.ph + a, wi = wo * d.sw - d.pw + b;
        if (hi >= 0 && hi < d.H && wi >= 0 && wi < d.W)
          v[t] = __ldg(reinterpret_cast<const uint4*>(x + (((int64_t)n * d.H + hi) * d.W + wi) * d.C) + g);
      }
    }
    float acc[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[j] = d.b >= 0 ? __ldg(p.params + d.b + g * 8 + j) : 0.f;
#pragma unroll
    for (int t = 0; t < kMaxTaps; ++t) {
      if (t < taps) {
        const uint32_t uw[4] = {v[t].x, v[t].y, v[t].z, v[t].w};
        // weights in [tap][C] order (d.w2): two float4 per tap and 8-channel group
        const float4* w4 = reinterpret_cast<const float4*>(p.params + d.w2 + t * d.C + g * 8);
        const float4 wa = __ldg(w4), wb = __ldg(w4 + 1);
        const float wv[8] = {wa.x, wa.y, wa.z, wa.w, wb.x, wb.y, wb.z, wb.w};
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const float xv = __uint_as_float(j & 1 ? (uw[j / 2] & 0xFFFF0000u) : (uw[j / 2] << 16));
          acc[j] = fmaf(xv, wv[j], acc[j]);
        }
      }
    }
    uint4 pk;
    __nv_bfloat162 h0v = __floats2bfloat162_rn(acc[0], acc[1]), h1v = __floats2bfloat162_rn(acc[2], acc[3]);
    __nv_bfloat162 h2v = __floats2bfloat162_rn(acc[4], acc[5]), h3v = __floats2bfloat162_rn(acc[6], acc[7]);
    pk.x = *reinterpret_cast<uint32_t*>(&h0v);
    pk.y = *reinterpret_cast<uint32_t*>(&h1v);
    pk.z = *reinterpret_cast<uint32_t*>(&h2v);
    pk.w = *reinterpret_cast<uint32_t*>(&h3v);
    reinterpret_cast<uint4*>(y + ((int64_t)row * d.Wo + wo) * d.C)[g] = pk;
  }
}

// ---------------------------------------------------------------------------
// direct NHWC convolution: one thread per output element, output channel
// fastest so a warp shares its input pixels (broadcast loads)
// ---------------------------------------------------------------------------
__global__ void conv_kernel(ConvDesc d, RunPtrs p) {
  const void* x = loc_ptr(d.x, p);
  void* y = const_cast<void*>(loc_ptr(d.y, p));
  const int cg = d.C / d.groups, kg = d.K / d.groups;
  const int64_t total = (int64_t)d.N * d.Ho * d.Wo * d.K;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int k = (int)(i % d.K);
    const int64_t pix = i / d.K;
    const int wo = (int)(pix % d.Wo);
    const int64_t t = pix / d.Wo;
    const int ho = (int)(t % d.Ho);
    const int n = (int)(t / d.Ho);
    const int g = k / kg;
    float acc = d.b >= 0 ? p.params[d.b + k] : 0.f;
    const float* w = p.params + d.w + (int64_t)k * d.kh * d.kw * cg;
    for (int a = 0; a < d.kh; ++a) {
      const int hi = ho * d.sh - d.ph + a;
      if (hi < 0 || hi >= d.H) continue;
      for (int b = 0; b < d.kw; ++b) {
        const int wi = wo * d.sw - d.pw + b;
        if (wi < 0 || wi >= d.W) continue;
        const int64_t base = (((int64_t)n * d.H + hi) * d.W + wi) * d.C + (int64_t)g * cg;
        const float* wr = w + (a * d.kw + b) * cg;
        for (int c = 0; c < cg; ++c) acc = fmaf(wr[c], ldv(x, base + c, d.x.dtype), acc);
      }
    }
    stv(y, i, acc, d.y.dtype);
  }
}

// ---------------------------------------------------------------------------
// elementwise, pooling, concat and GAP as standalone steps
// ---------------------------------------------------------------------------
__global__ void ew_kernel(EwDesc d, RunPtrs p) {
  void* y = const_cast<void*>(loc_ptr(d.y, p));
  const int64_t total = (int64_t)d.N * d.Ho * d.Wo * d.C;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int c = (int)(i % d.C);
    const int64_t pix = i / d.C;
    float v = 0.f;
    switch (d.kind) {
      case EW_BN:
        v = p.params[d.scale + c] * ldv(loc_ptr(d.x[0], p), i, d.x[0].dtype) + p.params[d.shift + c];
        break;
      case EW_RELU:
        v = fmaxf(ldv(loc_ptr(d.x[0], p), i, d.x[0].dtype), 0.f);
        break;
      case EW_SILU: {
        const float u = ldv(loc_ptr(d.x[0], p), i, d.x[0].dtype);
        v = u / (1.f + __expf(-u));
        break;
      }
      case EW_ADD:
        for (int j = 0; j < d.n_in; ++j) v += ldv(loc_ptr(d.x[j], p), i, d.x[j].dtype);
        break;
      case EW_CONCAT: {
        int cc = c, j = 0;
        while (cc >= d.xc[j]) cc -= d.xc[j++];
        v = ldv(loc_ptr(d.x[j], p), pix * d.xc[j] + cc, d.x[j].dtype);
        break;
      }
      case EW_MAXPOOL:
      case EW_AVGPOOL: {
        const int wo = (int)(pix % d.Wo);
        const int64_t t = pix / d.Wo;
        const int ho = (int)(t % d.Ho);
        const int n = (int)(t / d.Ho);
        const void* x = loc_ptr(d.x[0], p);
        float m = d.kind == EW_MAXPOOL ? -FLT_MAX : 0.f;
        for (int a = 0; a < d.k; ++a) {
          const int hi = ho * d.s - d.p + a;
          if (hi < 0 || hi >= d.H) continue;
          for (int b = 0; b < d.k; ++b) {
            const int wi = wo * d.s - d.p + b;
            if (wi < 0 || wi >= d.W) continue;
            const float u = ldv(x, (((int64_t)n * d.H + hi) * d.W + wi) * d.C + c, d.x[0].dtype);
            m = d.kind == EW_MAXPOOL ? fmaxf(m, u) : m + u;
          }
        }
        v = d.kind == EW_MAXPOOL ? m : m / (float)(d.k * d.k);
        break;
      }
      case EW_GAP: {
        const int n = (int)pix;   // Ho = Wo = 1
        const void* x = loc_ptr(d.x[0], p);
        float s = 0.f;
        for (int q = 0; q < d.H * d.W; ++q) s += ldv(x, ((int64_t)n * d.H * d.W + q) * d.C + c, d.x[0].dtype);
        v = s / (float)(d.H * d.W);
        break;
      }
    }
    stv(y, i, v, d.y.dtype);
  }
}

// bf16 NHWC, C % 8 == 0: the same per-element arithmetic as ew_kernel (same fp32 formula and
// summation order, same rounding), 8 channels per thread through 16-byte loads / stores -- the
// standalone BN / ReLU / SiLU / add / concat / pool steps of unfused (ablation) plans are
// HBM-bound and ew_kernel's 2-byte accesses reach a small fraction of the bandwidth
__device__ __forceinline__ void unpack8(const uint4& u, float* f) {
  const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const float2 t = __bfloat1622float2(h[j]);
    f[2 * j] = t.x;
    f[2 * j + 1] = t.y;
  }
}

__global__ void __launch_bounds__(256) ew_vec_kernel(EwDesc d, RunPtrs p) {
  uint4* y = reinterpret_cast<uint4*>(const_cast<void*>(loc_ptr(d.y, p)));
  const int cv = d.C / 8;
  const int64_t total = (int64_t)d.N * d.Ho * d.Wo * cv;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int c = (int)(i % cv) * 8;
    const int64_t pix = i / cv;
    float v[8], u[8];
    switch (d.kind) {
      case EW_BN:
        unpack8(reinterpret_cast<const uint4*>(loc_ptr(d.x[0], p))[i], u);
#pragma unroll
        for (int j = 0; j < 8; ++j) v[j] = p.params[d.scale + c + j] * u[j] + p.params[d.shift + c + j];
        break;
      case EW_RELU:
        unpack8(reinterpret_cast<const uint4*>(loc_ptr(d.x[0], p))[i], u);
#pragma unroll
        for (int j = 0; j < 8; ++j) v[j] = fmaxf(u[j], 0.f);
        break;
      case EW_SILU:
        unpack8(reinterpret_cast<const uint4*>(loc_ptr(d.x[0], p))[i], u);
#pragma unroll
        for (int j = 0; j < 8; ++j) v[j] = u[j] / (1.f + __expf(-u[j]));
        break;
      case EW_ADD:
#pragma unroll
        for (int j = 0; j < 8; ++j) v[j] = 0.f;
        for (int k = 0; k < d.n_in; ++k) {
          unpack8(reinterpret_cast<const uint4*>(loc_ptr(d.x[k], p))[i], u);
#pragma unroll
          for (int j = 0; j < 8; ++j) v[j] += u[j];
        }
        break;
      case EW_CONCAT: {
        int cc = c, k = 0;
        while (cc >= d.xc[k]) cc -= d.xc[k++];
        unpack8(reinterpret_cast<const uint4*>(loc_ptr(d.x[k], p))[(pix * d.xc[k] + cc) / 8], v);
        break;
      }
      case EW_MAXPOOL:
      case EW_AVGPOOL: {
        const int wo = (int)(pix % d.Wo);
        const int64_t t = pix / d.Wo;
        const int ho = (int)(t % d.Ho);
        const int n = (int)(t / d.Ho);
        const uint4* x = reinterpret_cast<const uint4*>(loc_ptr(d.x[0], p));
#pragma unroll
        for (int j = 0; j < 8; ++j) v[j] = d.kind == EW_MAXPOOL ? -FLT_MAX : 0.f;
        for (int a = 0; a < d.k; ++a) {
          const int hi = ho * d.s - d.p + a;
          if (hi < 0 || hi >= d.H) continue;
          for (int b = 0; b < d.k; ++b) {
            const int wi = wo * d.s - d.p + b;
            if (wi < 0 || wi >= d.W) continue;
            unpack8(x[((((int64_t)n * d.H + hi) * d.W + wi) * d.C + c) / 8], u);
#pragma unroll
            for (int j = 0; j < 8; ++j) v[j] = d.kind == EW_MAXPOOL ? fmaxf(v[j], u[j]) : v[j] + u[j];
          }
        }
        if (d.kind == EW_AVGPOOL)
#pragma unroll
          for (int j = 0; j < 8; ++j) v[j] = v[j] / (float)(d.k * d.k);
        break;
      }
    }
    uint4 o;
    __nv_bfloat162* h = reinterpret_cast<__nv_bfloat162*>(&o);
#pragma unroll
    for (int j = 0; j < 4; ++j) h[j] = __floats2bfloat162_rn(v[2 * j], v[2 * j + 1]);
    y[i] = o;
  }
}

// ---------------------------------------------------------------------------
// linear: SIMT tiled GEMM, 64x64 tile, 4x4 per thread
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(256) linear_kernel(LinearDesc d, RunPtrs p) {
  __shared__ float As[16][68];
  __shared__ float Bs[16][68];
  const void* x = loc_ptr(d.x, p);
  void* y = const_cast<void*>(loc_ptr(d.y, p));
  const float* Wt = p.params + d.w;
  const int m0 = blockIdx.y * 64, o0 = blockIdx.x * 64;
  const int tid = threadIdx.x, tx = tid % 16, ty = tid / 16;
  float acc[4][4] = {};
  for (int k0 = 0; k0 < d.K; k0 += 16) {
    for (int e = tid; e < 1024; e += 256) {
      const int r = e / 16, kk = e % 16;
      const int m = m0 + r, o = o0 + r, k = k0 + kk;
      As[kk][r] = (m < d.N && k < d.K) ? ldv(x, (int64_t)m * d.K + k, d.x.dtype) : 0.f;
      Bs[kk][r] = (o < d.O && k < d.K) ? Wt[(int64_t)o * d.K + k] : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < 16; ++kk) {
      float a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) a[i] = As[kk][ty * 4 + i], b[i] = Bs[kk][tx * 4 + i];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int m = m0 + ty * 4 + i, o = o0 + tx * 4 + j;
      if (m < d.N && o < d.O) {
        float v = acc[i][j] + (d.b >= 0 ? p.params[d.b + o] : 0.f);
        if (d.relu) v = fmaxf(v, 0.f);
        stv(y, (int64_t)m * d.O + o, v, d.y.dtype);
      }
    }
}

// ---------------------------------------------------------------------------
// fused group, generic interpreter: value of node `id` at (n, h, w, c),
// evaluated straight from the group's reduced inputs
// ---------------------------------------------------------------------------
struct GCtx {
  const GNode* nodes;
  const int32_t* children;
  RunPtrs p;
};

__device__ float geval(const GCtx& g, int id, int n, int h, int w, int c) {
  const GNode& nd = g.nodes[id];
  switch (nd.op) {
    case G_LCONV: {
      const void* t = loc_ptr(nd.t, g.p);
      const int64_t base = (((int64_t)n * nd.tH + h) * nd.tW + w) * nd.R;
      const float* wr = g.p.params + nd.w + (int64_t)c * nd.R;
      float acc = nd.b >= 0 ? g.p.params[nd.b + c] : 0.f;
      if (nd.t.dtype == DT_BF16) {
        const __nv_bfloat16* tp = reinterpret_cast<const __nv_bfloat16*>(t) + base;
        for (int k = 0; k < nd.R; ++k) acc = fmaf(wr[k], __bfloat162float(tp[k]), acc);
      } else {
        const float* tp = reinterpret_cast<const float*>(t) + base;
        for (int k = 0; k < nd.R; ++k) acc = fmaf(wr[k], tp[k], acc);
      }
      return acc;
    }
    case G_EXT:
      return ldv(loc_ptr(nd.t, g.p), (((int64_t)n * nd.tH + h) * nd.tW + w) * nd.tC + c, nd.t.dtype);
    case G_AFFINE:
      return g.p.params[nd.w + c] * geval(g, g.children[nd.child], n, h, w, c) + g.p.params[nd.b + c];
    case G_RELU:
      return fmaxf(geval(g, g.children[nd.child], n, h, w, c), 0.f);
    case G_SILU: {
      const float u = geval(g, g.children[nd.child], n, h, w, c);
      return u / (1.f + __expf(-u));
    }
    case G_ADD: {
      float s = 0.f;
      for (int j = 0; j < nd.nin; ++j) s += geval(g, g.children[nd.child + j], n, h, w, c);
      return s;
    }
    case G_CONCAT: {
      int cc = c;
      for (int j = 0; j < nd.nin; ++j) {
        const int ch = g.children[nd.child + j];
        const int cj = g.nodes[ch].C;
        if (cc < cj) return geval(g, ch, n, h, w, cc);
        cc -= cj;
      }
      return 0.f;
    }
    case G_MAXPOOL:
    case G_AVGPOOL: {
      const int ch = g.children[nd.child];
      const GNode& cn = g.nodes[ch];
      float m = nd.op == G_MAXPOOL ? -FLT_MAX : 0.f;
      for (int a = 0; a < nd.k; ++a) {
        const int hi = h * nd.s - nd.p + a;
        if (hi < 0 || hi >= cn.H) continue;
        for (int b = 0; b < nd.k; ++b) {
          const int wi = w * nd.s - nd.p + b;
          if (wi < 0 || wi >= cn.W) continue;
          const float u = geval(g, ch, n, hi, wi, c);
          m = nd.op == G_MAXPOOL ? fmaxf(m, u) : m + u;
        }
      }
      return nd.op == G_MAXPOOL ? m : m / (float)(nd.k * nd.k);
    }
  }
  return 0.f;
}

constexpr int kGP = 32;    // pixels per block
constexpr int kGC = 64;    // channel chunk
constexpr int kGMaxAcc = 32;

// fconv / store roots: t tile [32 px x 64 ch] in smem, then out += F t
__global__ void __launch_bounds__(256) group_simt_kernel(GroupDesc d, GCtx g) {
  __shared__ float tile[kGP][kGC + 1];
  const int64_t npix = (int64_t)d.N * d.H * d.W;
  const int64_t p0 = (int64_t)blockIdx.x * kGP;
  const int tid = threadIdx.x;
  void* y = const_cast<void*>(loc_ptr(d.y, g.p));
  float acc[kGMaxAcc];
#pragma unroll
  for (int j = 0; j < kGMaxAcc; ++j) acc[j] = 0.f;
  const int pi = tid % kGP, og = tid / kGP;
  for (int c0 = 0; c0 < d.C; c0 += kGC) {
    for (int idx = tid; idx < kGP * kGC; idx += blockDim.x) {
      const int r = idx / kGC, cc = idx % kGC;
      const int64_t pix = p0 + r;
      const int c = c0 + cc;
      float v = 0.f;
      if (pix < npix && c < d.C) {
        const int w = (int)(pix % d.W);
        const int64_t t = pix / d.W;
        v = geval(g, d.tnode, (int)(t / d.H), (int)(t % d.H), w, c);
      }
      tile[r][cc] = v;
    }
    __syncthreads();
    if (d.root == ROOT_FCONV) {
      const int cw = min(kGC, d.C - c0);
#pragma unroll
      for (int j = 0; j < kGMaxAcc; ++j) {
        const int o = og + 8 * j;
        if (o < d.Nout) {
          const float* fr = g.p.params + d.F + (int64_t)o * d.C + c0;
          float s = acc[j];
          for (int cc = 0; cc < cw; ++cc) s = fmaf(fr[cc], tile[pi][cc], s);
          acc[j] = s;
        }
      }
    } else {
      for (int idx = tid; idx < kGP * kGC; idx += blockDim.x) {
        const int r = idx / kGC, cc = idx % kGC;
        const int64_t pix = p0 + r;
        if (pix < npix && c0 + cc < d.C) stv(y, pix * d.C + c0 + cc, tile[r][cc], d.y.dtype);
      }
    }
    __syncthreads();
  }
  if (d.root == ROOT_FCONV) {
    const int64_t pix = p0 + pi;
    if (pix < npix) {
#pragma unroll
      for (int j = 0; j < kGMaxAcc; ++j) {
        const int o = og + 8 * j;
        if (o < d.Nout) stv(y, pix * d.Nout + o, acc[j] + (d.Fb >= 0 ? g.p.params[d.Fb + o] : 0.f), d.y.dtype);
      }
    }
  }
}

// GAP root: thread per (image, channel), fixed summation order (deterministic)
__global__ void group_gap_kernel(GroupDesc d, GCtx g) {
  const int n = blockIdx.y;
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= d.C) return;
  float s = 0.f;
  for (int h = 0; h < d.H; ++h)
    for (int w = 0; w < d.W; ++w) s += geval(g, d.tnode, n, h, w, c);
  stv(const_cast<void*>(loc_ptr(d.y, g.p)), (int64_t)n * d.C + c, s / (float)(d.H * d.W), d.y.dtype);
}

}  // namespace

void launch_conv(const ConvDesc& d, const RunPtrs& p, cudaStream_t s) {
  const int64_t total = (int64_t)d.N * d.Ho * d.Wo * d.K;
  conv_kernel<<<grid_for(total, 256), 256, 0, s>>>(d, p);
}

// transposed convolution: y[n, oh, ow, o] = b[o] + sum over taps (i, j) with oh = ih*sh - ph + i,
// ow = iw*sw - pw + j of sum_c x[n, ih, iw, c] W[c, o, i, j]; weights packed [i*kw + j][o][c].
// One thread per output element; the stride-2, 2x2 up-conv cores of UNet meet one tap each.
__global__ void conv_transpose_kernel(ConvDesc d, RunPtrs p) {
  const void* x = loc_ptr(d.x, p);
  void* y = const_cast<void*>(loc_ptr(d.y, p));
  const float* w = p.params + d.w;
  const int64_t total = (int64_t)d.N * d.Ho * d.Wo * d.K;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total; idx += (int64_t)gridDim.x * blockDim.x) {
    const int o = (int)(idx % d.K);
    int64_t r = idx / d.K;
    const int ow = (int)(r % d.Wo);
    r /= d.Wo;
    const int oh = (int)(r % d.Ho);
    const int n = (int)(r / d.Ho);
    float acc = d.b >= 0 ? p.params[d.b + o] : 0.f;
    for (int i = 0; i < d.kh; ++i) {
      const int th = oh + d.ph - i;
      if (th < 0 || th % d.sh) continue;
      const int ih = th / d.sh;
      if (ih >= d.H) continue;
      for (int j = 0; j < d.kw; ++j) {
        const int tw = ow + d.pw - j;
        if (tw < 0 || tw % d.sw) continue;
        const int iw = tw / d.sw;
        if (iw >= d.W) continue;
        const int64_t xb = (((int64_t)n * d.H + ih) * d.W + iw) * d.C;
        const float* wr = w + ((int64_t)(i * d.kw + j) * d.K + o) * d.C;
        for (int c = 0; c < d.C; ++c) acc += ldv(x, xb + c, d.x.dtype) * wr[c];
      }
    }
    stv(y, idx, acc, d.y.dtype);
  }
}

void launch_conv_transpose(const ConvDesc& d, const RunPtrs& p, cudaStream_t s) {
  const int64_t total = (int64_t)d.N * d.Ho * d.Wo * d.K;
  conv_transpose_kernel<<<grid_for(total, 256), 256, 0, s>>>(d, p);
}

bool dwconv_vec_ok(const ConvDesc& d) {
  return d.groups == d.C && d.K == d.C && d.C % 8 == 0 && d.x.dtype == DT_BF16 && d.y.dtype == DT_BF16 && d.w2 >= 0 &&
         d.kh * d.kw <= 9;
}

// ---------------------------------------------------------------------------
// CP depthwise core pair (reading R34): out(h, w, c) = sum_i Kv[c][i] sum_j Kh[c][j]
// x(h sv + i - pv, w sh + j - ph, c), zero outside the image -- the separable product of the
// K x 1 and 1 x K cores, whose intermediate (the K x 1 output) is never stored.
// ---------------------------------------------------------------------------
constexpr int kPairRows = 8;   // output rows per thread strip (fast kernel)

__device__ __forceinline__ void hcomb(float (&hv)[8], const uint4& l, const uint4& c, const uint4& r,
                                      const float (&kh)[3][8]) {
  const uint32_t ul[4] = {l.x, l.y, l.z, l.w}, uc[4] = {c.x, c.y, c.z, c.w}, ur[4] = {r.x, r.y, r.z, r.w};
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    const int q = j / 2;
    const bool hi = j & 1;
    const float xl = __uint_as_float(hi ? (ul[q] & 0xFFFF0000u) : (ul[q] << 16));
    const float xc = __uint_as_float(hi ? (uc[q] & 0xFFFF0000u) : (uc[q] << 16));
    const float xr = __uint_as_float(hi ? (ur[q] & 0xFFFF0000u) : (ur[q] << 16));
    hv[j] = fmaf(kh[0][j], xl, fmaf(kh[1][j], xc, kh[2][j] * xr));
  }
}

__device__ __forceinline__ uint4 shfl4(unsigned mask, const uint4& v, int delta, bool up) {
  uint4 o;
  if (up) {
    o.x = __shfl_up_sync(mask, v.x, delta); o.y = __shfl_up_sync(mask, v.y, delta);
    o.z = __shfl_up_sync(mask, v.z, delta); o.w = __shfl_up_sync(mask, v.w, delta);
  } else {
    o.x = __shfl_down_sync(mask, v.x, delta); o.y = __shfl_down_sync(mask, v.y, delta);
    o.z = __shfl_down_sync(mask, v.z, delta); o.w = __shfl_down_sync(mask, v.w, delta);
  }
  return o;
}

// fast path: bf16, C % 8 == 0 (<= 128 channels), K = 3, unit strides, pad 1, no biases.  A
// thread owns one (column, 8-channel group) and a strip of kPairRows output rows: it loads its
// own column's kPairRows + 2 input rows (16 bytes each, all in flight), takes the left / right
// neighbour columns from the lanes cg away (warp shuffles; lanes whose neighbour lies outside
// the warp load it), forms the horizontal 1 x 3 combination H of every input row and the
// vertical 3 x 1 combination of three H rows per output row.  x is read from HBM once and the
// output written once; the K x 1 intermediate never exists.
__global__ void __launch_bounds__(256, 2) dwpair_kernel(DwPairDesc d, RunPtrs p) {
  const __nv_bfloat16* x = reinterpret_cast<const __nv_bfloat16*>(loc_ptr(d.x, p));
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(const_cast<void*>(loc_ptr(d.y, p)));
  const int cg = d.C / 8;
  const int per_row = d.W * cg;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  const bool valid = idx < per_row;                  // idle lanes stay for the shuffles
  const int wo = valid ? idx / cg : 0, g = valid ? idx - (idx / cg) * cg : 0;
  const int lane = threadIdx.x & 31;
  float kv[3][8], kh[3][8];
#pragma unroll
  for (int j = 0; j < 8; ++j)
#pragma unroll
    for (int t = 0; t < 3; ++t) {
      kv[t][j] = __ldg(p.params + d.wv + (int64_t)(g * 8 + j) * 3 + t);
      kh[t][j] = __ldg(p.params + d.wh + (int64_t)(g * 8 + j) * 3 + t);
    }
  pdl_wait();
  pdl_trigger_early();
  const int spi = (d.Ho + kPairRows - 1) / kPairRows;
  const bool own_left = lane < cg, own_right = lane + cg >= 32;   // neighbour outside the warp
  const uint4 z = make_uint4(0, 0, 0, 0);
  for (int st = blockIdx.y; st < d.N * spi; st += gridDim.y) {
    const int n = st / spi, h0 = (st - n * spi) * kPairRows;
    const uint4* img = reinterpret_cast<const uint4*>(x + (int64_t)n * d.H * d.W * d.C);
    uint4 v[kPairRows + 2];
#pragma unroll
    for (int r = 0; r < kPairRows + 2; ++r) {
      const int hi = h0 - 1 + r;
      v[r] = (valid && hi >= 0 && hi < d.H && h0 + r - 2 < d.Ho) ? __ldg(img + ((int64_t)hi * d.W + wo) * cg + g) : z;
    }
    float ha[8], hb[8];
#pragma unroll
    for (int r = 0; r < kPairRows + 2; ++r) {
      const int hi = h0 - 1 + r;
      uint4 l = shfl4(0xffffffffu, v[r], cg, true), rr = shfl4(0xffffffffu, v[r], cg, false);
      const bool rowok = valid && hi >= 0 && hi < d.H;
      if (own_left) l = (rowok && wo > 0) ? __ldg(img + ((int64_t)hi * d.W + wo - 1) * cg + g) : z;
      if (own_right) rr = (rowok && wo + 1 < d.W) ? __ldg(img + ((int64_t)hi * d.W + wo + 1) * cg + g) : z;
      if (wo == 0) l = z;
      if (wo + 1 >= d.W) rr = z;
      float hc[8];
      hcomb(hc, l, v[r], rr, kh);
      if (r >= 2) {
        const int h = h0 + r - 2;
        if (valid && h < d.Ho) {
          float o[8];
#pragma unroll
          for (int j = 0; j < 8; ++j) o[j] = fmaf(kv[0][j], ha[j], fmaf(kv[1][j], hb[j], kv[2][j] * hc[j]));
          uint4 pk;
          __nv_bfloat162 q0 = __floats2bfloat162_rn(o[0], o[1]), q1 = __floats2bfloat162_rn(o[2], o[3]);
          __nv_bfloat162 q2 = __floats2bfloat162_rn(o[4], o[5]), q3 = __floats2bfloat162_rn(o[6], o[7]);
          pk.x = *reinterpret_cast<uint32_t*>(&q0);
          pk.y = *reinterpret_cast<uint32_t*>(&q1);
          pk.z = *reinterpret_cast<uint32_t*>(&q2);
          pk.w = *reinterpret_cast<uint32_t*>(&q3);
          reinterpret_cast<uint4*>(y + (((int64_t)n * d.Ho + h) * d.Wo + wo) * d.C)[g] = pk;
        }
      }
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        ha[j] = hb[j];
        hb[j] = hc[j];
      }
    }
  }
}

// any dtype / K / strides / biases: one thread per output element, the vertical core evaluated
// (with its bias) at each of the K columns the horizontal core reads
__global__ void __launch_bounds__(256) dwpair_generic_kernel(DwPairDesc d, RunPtrs p) {
  const void* x = loc_ptr(d.x, p);
  void* y = const_cast<void*>(loc_ptr(d.y, p));
  pdl_wait();
  const int64_t total = (int64_t)d.N * d.Ho * d.Wo * d.C;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int c = (int)(i % d.C);
    int64_t t = i / d.C;
    const int wo = (int)(t % d.Wo);
    t /= d.Wo;
    const int h = (int)(t % d.Ho);
    const int n = (int)(t / d.Ho);
    float acc = d.bh >= 0 ? p.params[d.bh + c] : 0.f;
    for (int j = 0; j < d.K; ++j) {
      const int w1 = wo * d.sh - d.ph + j;          // column of the vertical core's output
      if (w1 < 0 || w1 >= d.W) continue;
      float v = d.bv >= 0 ? p.params[d.bv + c] : 0.f;
      for (int q = 0; q < d.K; ++q) {
        const int r = h * d.sv - d.pv + q;
        if (r < 0 || r >= d.H) continue;
        v = fmaf(p.params[d.wv + (int64_t)c * d.K + q], ldv(x, (((int64_t)n * d.H + r) * d.W + w1) * d.C + c, d.x.dtype), v);
      }
      acc = fmaf(p.params[d.wh + (int64_t)c * d.K + j], v, acc);
    }
    stv(y, i, acc, d.y.dtype);
  }
}

bool dwpair_fast_ok(const DwPairDesc& d) {
  return d.x.dtype == DT_BF16 && d.y.dtype == DT_BF16 && d.C % 8 == 0 && d.C / 8 <= 16 && d.K == 3 && d.sv == 1 &&
         d.sh == 1 && d.pv == 1 && d.ph == 1 && d.bv < 0 && d.bh < 0 && d.Ho == d.H && d.Wo == d.W;
}

void launch_dwpair(const DwPairDesc& d, const RunPtrs& p, cudaStream_t s) {
  if (dwpair_fast_ok(d)) {
    const int xb = (d.W * (d.C / 8) + 255) / 256;
    const int strips = d.N * ((d.Ho + kPairRows - 1) / kPairRows);
    launch_pdl(dwpair_kernel, dim3((unsigned)xb, (unsigned)std::min(strips, std::max(1, 148 * 8 / xb))), dim3(256), 0, s,
               d, p);
    return;
  }
  const int64_t total = (int64_t)d.N * d.Ho * d.Wo * d.C;
  const int grid = (int)std::min<int64_t>((total + 255) / 256, 148LL * 16);
  launch_pdl(dwpair_generic_kernel, dim3(grid), dim3(256), 0, s, d, p);
}

void launch_dwconv_vec(const ConvDesc& d, const RunPtrs& p, cudaStream_t s) {
  const int per_row = d.Wo * (d.C / 8);
  const int rows = d.N * d.Ho;
  // rows per block: a persistent-ish y grid (8 blocks per SM per x chunk) instead of one
  // tiny block per output row
  const int xb = (per_row + 255) / 256;
  dim3 grid((unsigned)xb, (unsigned)std::min(rows, std::max(1, 148 * 8 / xb)));
  if (d.kh == 3 && d.kw == 1 && d.sh == 1 && d.sw == 1 && d.pw == 0 && d.Ho == d.H + 2 * d.ph - 2) {
    const int strips = d.N * ((d.Ho + kColRows - 1) / kColRows);
    launch_pdl(dwconv_col_kernel, dim3((unsigned)xb, (unsigned)std::min(strips, std::max(1, 148 * 8 / xb))), dim3(256), 0, s, d, p);
  } else if (d.kh == 3 && d.kw == 1)
    launch_pdl(dwconv_vec_kernel<3, 1>, grid, dim3(256), 0, s, d, p);
  else if (d.kh == 1 && d.kw == 3 && d.sh == 1 && d.sw == 1 && d.ph == 0 && d.pw == 1 && d.Wo == d.W &&
           d.Ho == d.H && d.C / 8 <= 16) {
    launch_pdl(dwconv_row_kernel, dim3((unsigned)xb, (unsigned)std::min((rows + 3) / 4, std::max(1, 148 * 8 / xb))), dim3(256), 0, s, d, p);
  } else if (d.kh == 1 && d.kw == 3)
    launch_pdl(dwconv_vec_kernel<1, 3>, grid, dim3(256), 0, s, d, p);
  else
    launch_pdl(dwconv_vec_kernel<0, 0>, grid, dim3(256), 0, s, d, p);
}

bool conv_rank_ok(const ConvDesc& d) {
  if (d.groups != 1 || d.x.dtype != DT_BF16 || d.y.dtype != DT_BF16) return false;
  // measured on B200 against the tcgen05 implicit GEMM (kernels_conv.cu): the
  // direct kernel wins while one 8-channel output group covers the layer
  if (d.C % 8 || d.C > 64 || d.K != 8) return false;
  return rank_tile(d).smem <= 160 * 1024;
}

void launch_conv_rank(const ConvDesc& d, const RunPtrs& p, cudaStream_t s) {
  static bool configured = false;
  if (!configured) {
    cudaFuncSetAttribute(conv_rank_kernel<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 160 * 1024);
    cudaFuncSetAttribute(conv_rank_kernel<16>, cudaFuncAttributeMaxDynamicSharedMemorySize, 160 * 1024);
    configured = true;
  }
  const RankTile t = rank_tile(d);
  dim3 grid((unsigned)(t.tiles_n * t.tiles_h * t.tiles_w), (unsigned)(d.K / t.kc));
  if (t.kc == 8)
    launch_pdl(conv_rank_kernel<8>, grid, dim3(256), t.smem, s, d, t, p);
  else
    launch_pdl(conv_rank_kernel<16>, grid, dim3(256), t.smem, s, d, t, p);
}

bool conv_small_ok(const ConvDesc& d) {
  return d.groups == 1 && d.C <= 8 && d.K <= 64 && d.sh == d.sw && d.sh <= 4 && conv_small_smem(d) <= 96 * 1024;
}

void launch_conv_small(const ConvDesc& d, const RunPtrs& p, cudaStream_t s) {
  static bool configured = false;
  if (!configured) {
    cudaFuncSetAttribute(conv_small_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 96 * 1024);
    configured = true;
  }
  const int tw = (d.Wo + kSmTW - 1) / kSmTW, th = (d.Ho + kSmTH - 1) / kSmTH;
  dim3 grid((unsigned)(d.N * tw * th), (unsigned)((d.K + kSmKC - 1) / kSmKC));
  conv_small_kernel<<<grid, 256, conv_small_smem(d), s>>>(d, p, tw, th);
}

static bool ew_vec_ok(const EwDesc& d, const RunPtrs& p) {
  if (d.kind == EW_GAP || d.C % 8 || d.y.dtype != DT_BF16 || ((uintptr_t)loc_ptr(d.y, p) & 15)) return false;
  for (int j = 0; j < d.n_in; ++j)
    if (d.x[j].dtype != DT_BF16 || ((uintptr_t)loc_ptr(d.x[j], p) & 15) || (d.kind == EW_CONCAT && d.xc[j] % 8))
      return false;
  return !getenv("TEMCO_NO_EW_VEC");
}

void launch_ew(const EwDesc& d, const RunPtrs& p, cudaStream_t s) {
  const int64_t total = (int64_t)d.N * d.Ho * d.Wo * d.C;
  if (ew_vec_ok(d, p)) {
    ew_vec_kernel<<<grid_for(total / 8, 256), 256, 0, s>>>(d, p);
    return;
  }
  ew_kernel<<<grid_for(total, 256), 256, 0, s>>>(d, p);
}

void launch_linear(const LinearDesc& d, const RunPtrs& p, cudaStream_t s) {
  dim3 grid((d.O + 63) / 64, (d.N + 63) / 64);
  linear_kernel<<<grid, 256, 0, s>>>(d, p);
}

void launch_group_simt(const GroupDesc& d, const GNode* nodes, const int32_t* children, const RunPtrs& p,
                       cudaStream_t s) {
  GCtx g{nodes, children, p};
  if (d.root == ROOT_GAP) {
    dim3 grid((d.C + 127) / 128, d.N);
    group_gap_kernel<<<grid, 128, 0, s>>>(d, g);
  } else {
    const int64_t npix = (int64_t)d.N * d.H * d.W;
    group_simt_kernel<<<(unsigned)((npix + kGP - 1) / kGP), 256, 0, s>>>(d, g);
  }
}

}  // namespace temco
