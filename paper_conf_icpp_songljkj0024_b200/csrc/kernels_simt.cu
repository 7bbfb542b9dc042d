// Generic SIMT kernels (fp32 arithmetic on fp32 / bf16 NHWC storage).
//
// These cover every step shape the planner can emit and are the fp32-mode
// path (no TF32: reading R22, the 1e-4 parity bar).  The tcgen05 kernels in
// kernels_tc.cu replace the hot fused groups in bf16 mode.
#include <cuda_bf16.h>

#include <cfloat>

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

void launch_ew(const EwDesc& d, const RunPtrs& p, cudaStream_t s) {
  const int64_t total = (int64_t)d.N * d.Ho * d.Wo * d.C;
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
