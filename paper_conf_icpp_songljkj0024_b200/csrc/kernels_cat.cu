// Register-resident fused kernel for single-level concat groups on mma.sync
// (bf16 mode): DenseNet's per-layer groups
//     fconv( ReLU( BN( concat[ pool(stem restore) | avgpool(transition lconv) | lconv_1 | ... ] ) ) )
// (Fig. 9a: concat -> fconv as one block-diagonal restore into the
// same accumulator; P:L305-317 for the pooled member), SURVEY 8(a) row a6.
//
// The group is parsed into one level (chain_parse.h): plain terms (lconv rows,
// BN-folded), tap-accumulate terms (avgpool over a linear member, weights / k^2)
// and at most one max/avg-pooled non-linear member (evaluated per tap, then
// pooled, then the post-BN shift).  The host flattens the work of one 16-pixel
// output block into a unit list, identical for every block:
//     for each 64-channel chunk: for each (term, tap) reaching it: one unit
// and the kernel walks (block, unit) with the A fragments (the term's reduced
// input rows at the tap, gathered straight from global memory into registers)
// of the next two units in flight.  The restored 16 x 64 chunk lives in 32
// accumulator registers; after its last unit it gets the level ReLU and is
// re-packed in place as the A operand of the reduce GEMM (out += P F^T).
// Everything is HBM-bound: bytes per pixel = sum of the reduced inputs + out.
#include <cuda_bf16.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <set>

#include "chain_parse.h"
#include "kernels.h"

namespace temco {

namespace {
using namespace chainp;

uint16_t f2bf(float f) {
  uint32_t u;
  memcpy(&u, &f, 4);
  u += 0x7FFF + ((u >> 16) & 1);
  return (uint16_t)(u >> 16);
}

}  // namespace

bool mma_cat_lower(const IR& ir, const Step& s, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                   CatDesc& d) {
  // roots: the fconv, or the fconvs of a merged group (reading R37) reading the same t
  std::vector<int> roots = {s.out};
  roots.insert(roots.end(), s.extra.begin(), s.extra.end());
  if (roots.size() > 4) return false;
  const int tsrc = ir.oin[s.out][0];
  int Nout = 0;
  for (int r : roots) {
    const Node& rn = ir.nodes[r];
    if (rn.role != ROLE_FCONV || rn.b || ir.oin[r].size() != 1 || ir.oin[r][0] != tsrc || rn.C % 8) return false;
    Nout += rn.C;
  }
  const Node& tn = ir.nodes[tsrc];
  const int C = tn.C;
  if (Nout % 8 || Nout > 64 || C % 8 || C > 64 * kCatMaxChunks) return false;
  const int Cpad = (C + 63) / 64 * 64;   // a short last chunk: zero weights / bias / F columns
  ChainParser P{ir, std::set<int>(s.members.begin(), s.members.end()), C, {}, tn.H, tn.W};
  for (int r : roots) P.members.erase(r);
  std::vector<PLevel> levels;
  if (!P.chain(tsrc, levels)) return false;
  if (P.visited != P.members || levels.size() != 1) return false;
  const PLevel& L = levels[0];
  if (L.pm.size() > 1) return false;
  const PMember* pm = L.pm.empty() ? nullptr : &L.pm[0];
  if (pm && (pm->c0 % 64 || pm->C % 64 || (pm->kind == 2 && pm->p != 0))) return false;

  d = CatDesc();
  d.C = C;
  d.nchunks = Cpad / 64;
  d.Nout = Nout;
  d.NO = Nout / 8;
  d.H = tn.H;
  d.W = tn.W;
  d.npix = ir.batch * tn.H * tn.W;
  if ((int64_t)ir.batch * tn.H * tn.W >= (1LL << 31) - 16) return false;
  d.nblocks = (d.npix + 15) / 16;
  d.relu = L.relu ? 1 : 0;
  d.n_out = (int)roots.size();
  d.ycol[0] = 0;
  for (int k = 0; k < d.n_out; ++k) {
    const Loc& yl = loc.at(roots[k]);
    if (yl.where != W_ARENA || yl.dtype != DT_BF16) return false;
    d.ys[k] = yl;
    d.ycol[k + 1] = d.ycol[k] + ir.nodes[roots[k]].C;
  }
  d.y = d.ys[0];

  std::vector<uint16_t> blob;
  std::vector<float> fbias;
  int64_t flops = 0, bytes = 0;
  // terms: plain / tap-accumulate (level), then the pooled member's
  auto add_term = [&](const PTerm& t, int kind) -> bool {
    if (d.n_terms == kCatMaxTerms) return false;
    const Node& lc = ir.nodes[t.lconv];
    const int r = ir.oin[t.lconv][0];
    const Node& rn = ir.nodes[r];
    const Loc& rl = loc.at(r);
    if (rl.where != W_ARENA || rl.dtype != DT_BF16 || rn.C % 8 || rn.C > 64 || lc.C % 8 || t.c0 % 8) return false;
    CatTerm& T = d.term[d.n_terms++];
    T.r = rl;
    T.R = rn.C;
    T.ks = (rn.C + 15) / 16;
    T.c0 = t.c0;
    T.C = lc.C;
    T.Hin = rn.H;
    T.Win = rn.W;
    T.kind = kind;
    if (kind == 0) {
      T.tk = t.tk;
      T.ts = t.ts;
      T.tp = t.tp;
    } else {
      T.tk = pm->k;
      T.ts = pm->s;
      T.tp = pm->p;
    }
    T.rs = T.ks * 16 + 8;
    while (blob.size() % 8) blob.push_back(0);
    T.w = (int32_t)blob.size();
    blob.resize(blob.size() + (size_t)lc.C * T.rs, 0);
    for (int c = 0; c < lc.C; ++c)
      for (int k = 0; k < T.R; ++k)
        blob[T.w + (size_t)c * T.rs + k] = f2bf((float)(t.scale[c] * (*lc.w)[(size_t)c * T.R + k]));
    const int64_t in_pix = (int64_t)ir.batch * rn.H * rn.W;
    flops += in_pix * 2LL * lc.C * T.R;
    bytes += in_pix * 2LL * T.R;
    return true;
  };
  for (const PTerm& t : L.terms)
    if (!add_term(t, 0)) return false;
  d.n_plain = d.n_terms;
  if (pm)
    for (const PTerm& t : pm->terms)
      if (!add_term(t, 1)) return false;
  // F [Nout][C + 8]
  while (blob.size() % 8) blob.push_back(0);
  d.f = (int32_t)blob.size();
  d.fs = Cpad + 8;
  blob.resize(blob.size() + (size_t)Nout * d.fs, 0);
  for (int k = 0; k < d.n_out; ++k) {   // the roots' F stacked row-wise
    const Node& rn = ir.nodes[roots[k]];
    for (int o = 0; o < rn.C; ++o)
      for (int c = 0; c < C; ++c) blob[d.f + (size_t)(d.ycol[k] + o) * d.fs + c] = f2bf((*rn.w)[(size_t)o * C + c]);
  }
  while (blob.size() % 8) blob.push_back(0);
  d.blob_bf16 = (int32_t)blob.size();
  // fp32: level bias [C] (pooled channels: the post-pool shift), member bias [C] (0 elsewhere)
  d.lbias = 0;
  d.mbias = Cpad;
  fbias.assign(2 * Cpad, 0.f);
  for (int c = 0; c < C; ++c) fbias[c] = (float)L.bias[c];
  if (pm) {
    for (int c = 0; c < pm->C; ++c) fbias[Cpad + pm->c0 + c] = (float)pm->bias[c];
    d.pool = pm->kind;
    d.pk = pm->k;
    d.ps = pm->s;
    d.pp = pm->p;
    d.mrelu = pm->relu ? 1 : 0;
    d.pc0 = pm->c0 / 64;
    d.pc1 = (pm->c0 + pm->C) / 64;
  }
  for (float b : fbias) {
    uint32_t u;
    memcpy(&u, &b, 4);
    blob.push_back((uint16_t)(u & 0xFFFF));
    blob.push_back((uint16_t)(u >> 16));
  }
  while (blob.size() % 8) blob.push_back(0);
  d.blob_bytes = (int32_t)blob.size() * 2;
  if (d.blob_bytes > 200 * 1024) return false;
  // unit list of one block
  std::vector<CatUnit> U;
  for (int ch = 0; ch < d.nchunks; ++ch) {
    const bool pooled = pm && ch >= d.pc0 && ch < d.pc1;
    const size_t first = U.size();
    auto hits = [&](const CatTerm& T, int& lo, int& hi) {
      lo = std::max(T.c0, ch * 64);
      hi = std::min(T.c0 + T.C, ch * 64 + 64);
      return lo < hi;
    };
    if (pooled) {
      const int taps = pm->k * pm->k;
      for (int tap = 0; tap < taps; ++tap) {
        const size_t tf = U.size();
        for (int j = d.n_plain; j < d.n_terms; ++j) {
          int lo, hi;
          if (!hits(d.term[j], lo, hi)) continue;
          CatUnit u{};
          u.term = (int16_t)j;
          u.tap = (int8_t)tap;
          u.chunk = (int16_t)ch;
          u.nt0 = (int8_t)((lo - ch * 64) / 8);
          u.nt1 = (int8_t)((hi - ch * 64) / 8);
          u.woff = d.term[j].w + (lo - d.term[j].c0) * d.term[j].rs;
          U.push_back(u);
        }
        if (U.size() == tf) return false;
        U[tf].flags |= CU_TAP_FIRST;
        U.back().flags |= CU_TAP_LAST;
      }
    } else {
      for (int j = 0; j < d.n_plain; ++j) {
        int lo, hi;
        if (!hits(d.term[j], lo, hi)) continue;
        for (int tap = 0; tap < d.term[j].tk * d.term[j].tk; ++tap) {
          CatUnit u{};
          u.term = (int16_t)j;
          u.tap = (int8_t)tap;
          u.chunk = (int16_t)ch;
          u.nt0 = (int8_t)((lo - ch * 64) / 8);
          u.nt1 = (int8_t)((hi - ch * 64) / 8);
          u.woff = d.term[j].w + (lo - d.term[j].c0) * d.term[j].rs;
          U.push_back(u);
        }
      }
      if (U.size() == first) {   // a chunk no term reaches (zero restore): one empty unit
        CatUnit u{};
        u.term = -1;
        u.chunk = (int16_t)ch;
        U.push_back(u);
      }
    }
    U[first].flags |= CU_FIRST;
    U.back().flags |= CU_LAST;
    if (pooled) U[first].flags |= CU_POOLED, U.back().flags |= CU_POOLED;
    for (size_t i = first; i < U.size(); ++i)
      if (pooled) U[i].flags |= CU_POOLED;
  }
  if ((int)U.size() > kCatMaxUnits) return false;
  d.n_units = (int)U.size();
  for (int c = 0, i = 0; c <= d.nchunks; ++c) {
    while (i < d.n_units && U[i].chunk < c) ++i;
    d.chunk_u0[c] = (int16_t)i;
  }
  for (int i = 0; i < d.n_units; ++i) d.unit[i] = U[i];
  while (tcw.size() % 512) tcw.push_back(0);
  d.blob = (int64_t)tcw.size();
  tcw.insert(tcw.end(), blob.begin(), blob.end());
  d.alg_flops = flops + (int64_t)d.npix * 2LL * Nout * C;
  d.alg_bytes = bytes + (int64_t)d.npix * 2LL * Nout;
  return true;
}

namespace {

constexpr int kCatWarps = 16;

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

// output-pixel coordinates of the two fragment rows of a block
struct CatRows {
  int n[2], ho[2], wo[2];
  bool ok[2];
};

__device__ __forceinline__ CatRows cat_rows(const CatDesc& d, int blk, int g) {
  CatRows r;
  const int hw = d.H * d.W;
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    const int m = blk * 16 + g + 8 * h;
    r.ok[h] = m < d.npix;
    r.n[h] = m / hw;
    const int rem = m - r.n[h] * hw;
    r.ho[h] = rem / d.W;
    r.wo[h] = rem - r.ho[h] * d.W;
  }
  return r;
}

// A fragments of one unit (term, tap) for the block's rows; also the rows'
// tap validity (max-pool masking)
template <int KSM>
__device__ __forceinline__ void cat_load(uint32_t (&a)[KSM][4], bool (&valid)[2], const CatDesc& d, const RunPtrs& p,
                                         const CatUnit& u, const CatRows& rw, int t4) {
  if (u.term < 0) {
#pragma unroll
    for (int ks = 0; ks < KSM; ++ks) a[ks][0] = a[ks][1] = a[ks][2] = a[ks][3] = 0u;
    valid[0] = valid[1] = false;
    return;
  }
  const CatTerm& T = d.term[u.term];
  const uint32_t* x = reinterpret_cast<const uint32_t*>(p.arena + T.r.off);
  const int ty = u.tap / T.tk, tx = u.tap - ty * T.tk;
  int64_t off[2];
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    const int hi = rw.ho[h] * T.ts - T.tp + ty, wi = rw.wo[h] * T.ts - T.tp + tx;
    valid[h] = rw.ok[h] && hi >= 0 && hi < T.Hin && wi >= 0 && wi < T.Win;
    off[h] = ((int64_t)(rw.n[h] * T.Hin + hi) * T.Win + wi) * (T.R / 2);
  }
#pragma unroll
  for (int ks = 0; ks < KSM; ++ks) {
    const int k0 = ks * 16 + 2 * t4, k1 = k0 + 8;
    a[ks][0] = (valid[0] && k0 < T.R) ? __ldg(x + off[0] + k0 / 2) : 0u;
    a[ks][1] = (valid[1] && k0 < T.R) ? __ldg(x + off[1] + k0 / 2) : 0u;
    a[ks][2] = (valid[0] && k1 < T.R) ? __ldg(x + off[0] + k1 / 2) : 0u;
    a[ks][3] = (valid[1] && k1 < T.R) ? __ldg(x + off[1] + k1 / 2) : 0u;
  }
}

template <int NO, int KSM, bool POOL>
__global__ void __launch_bounds__(32 * kCatWarps, 1) mma_cat_kernel(const __grid_constant__ CatDesc d, RunPtrs p,
                                                                     const uint16_t* __restrict__ tcw) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int g = lane / 4, t4 = lane % 4;
  {
    const uint4* src = reinterpret_cast<const uint4*>(tcw + d.blob);
    uint4* dst = reinterpret_cast<uint4*>(smem);
    for (int i = threadIdx.x; i < d.blob_bytes / 16; i += blockDim.x) dst[i] = __ldg(src + i);
  }
  __syncthreads();
  const __nv_bfloat16* blob = reinterpret_cast<const __nv_bfloat16*>(smem);
  const float* fb = reinterpret_cast<const float*>(smem + (size_t)d.blob_bf16 * 2);
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.arena + d.y.off);
  const int lq = lane >> 3, lr = lane & 7;
  const uint32_t sbase = s_u32(blob);
  const int nw = gridDim.x * kCatWarps;
  const int NU = d.n_units;
  // prefetch cursor: (block, unit) two units ahead of the compute cursor
  int pblk = blockIdx.x * kCatWarps + warp, pu = 0;
  CatRows prow = cat_rows(d, pblk, g);
  uint32_t a[KSM][4], an[KSM][4], ann[KSM][4];
  bool va[2], van[2], vann[2];
  auto pf_next = [&](uint32_t (&dst)[KSM][4], bool (&v)[2]) {
    if (pblk < d.nblocks) cat_load<KSM>(dst, v, d, p, d.unit[pu], prow, t4);
    if (++pu == NU) {
      pu = 0;
      pblk += nw;
      prow = cat_rows(d, pblk, g);
    }
  };
  pf_next(a, va);
  pf_next(an, van);
  float O[NO][4];
  float D[8][4], run[POOL ? 8 : 1][4];
  for (int blk = blockIdx.x * kCatWarps + warp; blk < d.nblocks; blk += nw) {
#pragma unroll
    for (int i = 0; i < NO; ++i) O[i][0] = O[i][1] = O[i][2] = O[i][3] = 0.f;
    for (int ui = 0; ui < NU; ++ui) {
      pf_next(ann, vann);
      const CatUnit u = d.unit[ui];
      const int c0 = u.chunk * 64;
      const bool pooled = POOL && (u.flags & CU_POOLED) != 0;
      if ((u.flags & CU_FIRST) && !pooled) {
#pragma unroll
        for (int nt = 0; nt < 8; ++nt) {
          const float2 b = *reinterpret_cast<const float2*>(fb + d.lbias + c0 + nt * 8 + 2 * t4);
          D[nt][0] = b.x; D[nt][1] = b.y; D[nt][2] = b.x; D[nt][3] = b.y;
        }
      }
      if (pooled && (u.flags & CU_TAP_FIRST)) {
#pragma unroll
        for (int nt = 0; nt < 8; ++nt) {
          const float2 b = *reinterpret_cast<const float2*>(fb + d.mbias + c0 + nt * 8 + 2 * t4);
          D[nt][0] = b.x; D[nt][1] = b.y; D[nt][2] = b.x; D[nt][3] = b.y;
        }
      }
      if (u.term >= 0) {
        const int nks = d.term[u.term].ks, rs = d.term[u.term].rs;
        // lane address of ldmatrix: rows (n-tile base + lr), k half lq & 1; x4 covers two n-tiles
        const uint32_t wb = sbase + (uint32_t)((u.woff + ((lq >> 1) * 8 + lr) * rs + (lq & 1) * 8) * 2);
        const uint32_t wb2 = sbase + (uint32_t)((u.woff + lr * rs + (lq & 1) * 8) * 2);
#pragma unroll
        for (int ks = 0; ks < KSM; ++ks) {
          if (ks < nks) {
#pragma unroll
            for (int nt = 0; nt < 8; nt += 2) {
              if (nt >= u.nt0 && nt < u.nt1) {
                const uint32_t roff = (uint32_t)(((nt - u.nt0) * 8 * rs + ks * 16) * 2);
                if (nt + 1 < u.nt1) {
                  uint32_t b0, b1, b2, b3;
                  ldsm_x4(wb + roff, b0, b1, b2, b3);
                  mma16816(D[nt], a[ks], b0, b1);
                  mma16816(D[nt + 1], a[ks], b2, b3);
                } else {
                  uint32_t b0, b1;
                  ldsm_x2(wb2 + roff, b0, b1);
                  mma16816(D[nt], a[ks], b0, b1);
                }
              } else if (nt + 1 >= u.nt0 && nt + 1 < u.nt1) {   // odd start: tile nt + 1 alone
                uint32_t b0, b1;
                ldsm_x2(wb2 + (uint32_t)(((nt + 1 - u.nt0) * 8 * rs + ks * 16) * 2), b0, b1);
                mma16816(D[nt + 1], a[ks], b0, b1);
              }
            }
          }
        }
      }
      if constexpr (POOL) if (pooled && (u.flags & CU_TAP_LAST)) {
        // member activation, max / sum over the pooling window (max: taps outside excluded)
        const int tap = u.tap;
        const float n0 = (d.pool == 1 && !va[0]) ? -INFINITY : 0.f;
        const float n1 = (d.pool == 1 && !va[1]) ? -INFINITY : 0.f;
#pragma unroll
        for (int nt = 0; nt < 8; ++nt)
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            float z = d.mrelu ? fmaxf(D[nt][i], 0.f) : D[nt][i];
            z += i < 2 ? n0 : n1;
            run[nt][i] = tap == 0 ? z : d.pool == 1 ? fmaxf(run[nt][i], z) : run[nt][i] + z;
          }
      }
      if (u.flags & CU_LAST) {
        if constexpr (POOL) if (pooled) {
          const float sc = d.pool == 2 ? 1.f / (float)(d.pk * d.pk) : 1.f;
#pragma unroll
          for (int nt = 0; nt < 8; ++nt) {
            const float2 b = *reinterpret_cast<const float2*>(fb + d.lbias + c0 + nt * 8 + 2 * t4);
            D[nt][0] = run[nt][0] * sc + b.x;
            D[nt][1] = run[nt][1] * sc + b.y;
            D[nt][2] = run[nt][2] * sc + b.x;
            D[nt][3] = run[nt][3] * sc + b.y;
          }
        }
        if (d.relu) {
#pragma unroll
          for (int nt = 0; nt < 8; ++nt)
#pragma unroll
            for (int i = 0; i < 4; ++i) D[nt][i] = fmaxf(D[nt][i], 0.f);
        }
        // reduce: O += P F^T over this chunk
#pragma unroll
        for (int kp = 0; kp < 2; ++kp) {
          uint32_t pa[2][4];
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int ks = 2 * kp + h;
            pa[h][0] = pk2(D[2 * ks][0], D[2 * ks][1]);
            pa[h][1] = pk2(D[2 * ks][2], D[2 * ks][3]);
            pa[h][2] = pk2(D[2 * ks + 1][0], D[2 * ks + 1][1]);
            pa[h][3] = pk2(D[2 * ks + 1][2], D[2 * ks + 1][3]);
          }
#pragma unroll
          for (int nb = 0; nb < NO; ++nb) {
            if (nb >= d.NO) break;   // NO is the template bound (even), d.NO the real n-tile count
            uint32_t f0, f1, f2, f3;
            ldsm_x4(sbase + (uint32_t)((d.f + (nb * 8 + lr) * d.fs + c0 + kp * 32 + lq * 8) * 2), f0, f1, f2, f3);
            mma16816(O[nb], pa[0], f0, f1);
            mma16816(O[nb], pa[1], f2, f3);
          }
        }
      }
#pragma unroll
      for (int ks = 0; ks < KSM; ++ks)
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          a[ks][i] = an[ks][i];
          an[ks][i] = ann[ks][i];
        }
      va[0] = van[0]; va[1] = van[1];
      van[0] = vann[0]; van[1] = vann[1];
    }
    const int m0 = blk * 16 + g, m1 = m0 + 8;
#pragma unroll
    for (int nb = 0; nb < NO; ++nb) {
      if (nb >= d.NO) break;
      const int col = nb * 8 + 2 * t4;
      if (m0 < d.npix) *reinterpret_cast<uint32_t*>(y + (int64_t)m0 * d.Nout + col) = pk2(O[nb][0], O[nb][1]);
      if (m1 < d.npix) *reinterpret_cast<uint32_t*>(y + (int64_t)m1 * d.Nout + col) = pk2(O[nb][2], O[nb][3]);
    }
  }
}

template <int NO, int KSM, bool POOL>
void launch_cat_t(const CatDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  static bool configured = false;
  static int sms = 148;
  if (!configured) {
    cudaFuncSetAttribute(mma_cat_kernel<NO, KSM, POOL>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    configured = true;
  }
  int per_sm = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, mma_cat_kernel<NO, KSM, POOL>, 32 * kCatWarps, d.blob_bytes);
  const int grid = std::min((d.nblocks + kCatWarps - 1) / kCatWarps, sms * std::max(per_sm, 1));
  mma_cat_kernel<NO, KSM, POOL><<<grid, 32 * kCatWarps, d.blob_bytes, s>>>(d, p, tcw);
}

// ---------------------------------------------------------------------------
// Pooled-concat groups whose pooled member is a 3x3 / stride-2 max pool over a
// rank <= 16 restore of 64 channels (the stem restore copies: ResNet-50's
// stem -> maxpool -> layer1 groups, DenseNet-121's block-1 layer groups).
// Restore-once: a CTA owns an 8 x 16 output tile; phase 1 restores every pixel
// of its (2*8+1) x (2*16+1) input footprint once (act(Lhat r + b), bf16, -inf
// outside the image) into SMEM -- 2.25 restores per output instead of the 9 of
// a per-tap evaluation; phase 2 max-pools each output's 3 x 3 window straight
// into the bf16x2 A fragments of the reduce GEMM, adds the post-pool shift and
// the level ReLU, then the plain concat terms (other 64-channel chunks) are
// restored from global memory per output block as in the generic kernel.
// ---------------------------------------------------------------------------
constexpr int kPcTH = 8, kPcTW = 16, kPcWarps = 8, kPcStride = 34;   // words per footprint pixel (64 bf16 ch + pad: conflict-free pooling reads)

template <int NO, int PK, int PS, int PP>   // pool window / stride / pad: (3, 2, 1) or (2, 2, 0)
__global__ void __launch_bounds__(32 * kPcWarps, 2) mma_poolcat_kernel(const __grid_constant__ CatDesc d, RunPtrs p,
                                                                    const uint16_t* __restrict__ tcw, int tiles_w,
                                                                    int tiles_h) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int g = lane / 4, t4 = lane % 4;
  {
    const uint4* src = reinterpret_cast<const uint4*>(tcw + d.blob);
    uint4* dst = reinterpret_cast<uint4*>(smem);
    for (int i = threadIdx.x; i < d.blob_bytes / 16; i += blockDim.x) dst[i] = __ldg(src + i);
  }
  __syncthreads();
  pdl_wait();
  pdl_trigger_early();
  const __nv_bfloat16* blob = reinterpret_cast<const __nv_bfloat16*>(smem);
  const float* fb = reinterpret_cast<const float*>(smem + (size_t)d.blob_bf16 * 2);
  uint32_t* fp = reinterpret_cast<uint32_t*>(smem + (d.blob_bytes + 15) / 16 * 16);   // footprint [PR*PC][kPcStride]
  const int lq = lane >> 3, lr = lane & 7;
  const uint32_t sbase = s_u32(blob);
  const CatTerm& M = d.term[d.n_plain];                 // the pooled member's (single) term
  const int PR = (kPcTH - 1) * PS + PK, PC = (kPcTW - 1) * PS + PK;
  // member restore fragments and bias (registers for the whole kernel)
  // 3x3 windows: the member's restore weights are ldmatrix'd from SMEM per use (holding them in 16
  // registers for the whole kernel spilled: local-memory loads and ~200 register moves per tile);
  // 2x2 windows (VGG) keep them in registers (measured faster there)
  constexpr bool kWmReg = PK == 2;
  uint32_t wm[kWmReg ? 8 : 1][2];
  if constexpr (kWmReg) {
#pragma unroll
    for (int np = 0; np < 4; ++np)
      ldsm_x4(sbase + (uint32_t)((M.w + (np * 16 + (lq >> 1) * 8 + lr) * M.rs + (lq & 1) * 8) * 2), wm[2 * np][0],
              wm[2 * np][1], wm[2 * np + 1][0], wm[2 * np + 1][1]);
  }
  float mb[8][2];
#pragma unroll
  for (int nt = 0; nt < 8; ++nt) {
    const float2 b = *reinterpret_cast<const float2*>(fb + d.mbias + nt * 8 + 2 * t4);
    mb[nt][0] = b.x;
    mb[nt][1] = b.y;
  }
  const uint32_t* rm = reinterpret_cast<const uint32_t*>(p.arena + M.r.off);
  const int ntiles = d.npix / (d.H * d.W) * tiles_w * tiles_h;
  for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int n = tile / (tiles_w * tiles_h);
    const int oh0 = (tile / tiles_w) % tiles_h * kPcTH, ow0 = tile % tiles_w * kPcTW;
    const int ih0 = oh0 * PS - PP, iw0 = ow0 * PS - PP;
    // ---- phase 1: restore the footprint once; all of the warp's loads first (in flight together)
    constexpr int kMaxB = 5;   // footprint blocks per warp: ceil(17 * 33 / 16 / 8)
    uint32_t a[kMaxB][4];
    bool v[kMaxB][2];
#pragma unroll
    for (int q = 0; q < kMaxB; ++q) {
      const int fb16 = warp + q * kPcWarps;
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int px = fb16 * 16 + g + 8 * h;
        const int fr = px / PC, fc = px - fr * PC;
        const int ih = ih0 + fr, iw = iw0 + fc;
        v[q][h] = px < PR * PC && ih >= 0 && ih < M.Hin && iw >= 0 && iw < M.Win;
        const int64_t off = ((int64_t)(n * M.Hin + ih) * M.Win + iw) * (M.R / 2);
        a[q][h] = (v[q][h] && 2 * t4 < M.R) ? __ldg(rm + off + t4) : 0u;
        a[q][2 + h] = (v[q][h] && 2 * t4 + 8 < M.R) ? __ldg(rm + off + t4 + 4) : 0u;
      }
    }
#pragma unroll
    for (int q = 0; q < kMaxB; ++q) {
      const int fb16 = warp + q * kPcWarps;
      if (fb16 * 16 >= PR * PC) break;
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) {
        float D[4] = {mb[nt][0], mb[nt][1], mb[nt][0], mb[nt][1]};
        uint32_t w0, w1;   // n-tile nt: rows 8 nt .. of the member's Lhat, k halves 0 / 1
        if constexpr (kWmReg) {
          w0 = wm[nt][0];
          w1 = wm[nt][1];
        } else {
          ldsm_x2(sbase + (uint32_t)((M.w + (nt * 8 + lr) * M.rs + (lq & 1) * 8) * 2), w0, w1);
        }
        mma16816(D, a[q], w0, w1);
        if (d.mrelu) {
#pragma unroll
          for (int i = 0; i < 4; ++i) D[i] = fmaxf(D[i], 0.f);
        }
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int px = fb16 * 16 + g + 8 * h;
          if (px < PR * PC)
            fp[px * kPcStride + nt * 4 + t4] = v[q][h] ? pk2(D[2 * h], D[2 * h + 1]) : 0xFF80FF80u;   // -inf pair
        }
      }
    }
    __syncthreads();
    // ---- phase 2: one 16-pixel output row per warp
    if (warp < kPcTH) {
      const int oh = oh0 + warp;
      float O[NO][4];
#pragma unroll
      for (int i = 0; i < NO; ++i) O[i][0] = O[i][1] = O[i][2] = O[i][3] = 0.f;
      CatRows rw;
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        rw.n[h] = n;
        rw.ho[h] = oh;
        rw.wo[h] = ow0 + g + 8 * h;
        rw.ok[h] = oh < d.H && rw.wo[h] < d.W;
      }
      // chunk 0: the pooled member -> P fragments (bf16x2 max over the 3 x 3 window)
#pragma unroll
      for (int ks = 0; ks < 4; ++ks) {
        uint32_t pa[4];
#pragma unroll
        for (int r4 = 0; r4 < 4; ++r4) {
          const int h = r4 & 1, chw = ks * 8 + t4 + (r4 >> 1) * 4;   // word of channels 16ks + 2t4 (+8)
          const int fc0 = PS * (g + 8 * h), fr0 = PS * warp;
          __nv_bfloat162 m = __halves2bfloat162(__float2bfloat16_rn(-INFINITY), __float2bfloat16_rn(-INFINITY));
#pragma unroll
          for (int ty = 0; ty < PK; ++ty)
#pragma unroll
            for (int tx = 0; tx < PK; ++tx) {
              const uint32_t w = fp[((fr0 + ty) * PC + fc0 + tx) * kPcStride + chw];
              m = __hmax2(m, *reinterpret_cast<const __nv_bfloat162*>(&w));
            }
          // + post-pool shift (the level bias of these channels), level ReLU
          const int ch = ks * 16 + (r4 >> 1) * 8 + 2 * t4;
          float lo = __low2float(m) + fb[d.lbias + ch], hi = __high2float(m) + fb[d.lbias + ch + 1];
          if (d.relu) lo = fmaxf(lo, 0.f), hi = fmaxf(hi, 0.f);
          pa[r4 == 0 ? 0 : r4 == 1 ? 1 : r4 == 2 ? 2 : 3] = pk2(lo, hi);
        }
#pragma unroll
        for (int nb = 0; nb < NO; ++nb) {
          if (nb >= d.NO) break;
          uint32_t f0, f1;
          ldsm_x2(sbase + (uint32_t)((d.f + (nb * 8 + lr) * d.fs + ks * 16 + (lq & 1) * 8) * 2), f0, f1);
          mma16816(O[nb], pa, f0, f1);
        }
      }
      // other chunks: plain concat terms, restored per output block
      for (int ch = 1; ch < d.nchunks; ++ch) {
        float D[8][4];
#pragma unroll
        for (int nt = 0; nt < 8; ++nt) {
          const float2 b = *reinterpret_cast<const float2*>(fb + d.lbias + ch * 64 + nt * 8 + 2 * t4);
          D[nt][0] = b.x; D[nt][1] = b.y; D[nt][2] = b.x; D[nt][3] = b.y;
        }
        // this chunk's units only, their A loads issued together (in flight at once)
        const int cu0 = d.chunk_u0[ch], cu1 = d.chunk_u0[ch + 1];
        for (int ub = cu0; ub < cu1; ub += 4) {
        uint32_t aq[4][1][4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          bool va[2];
          if (ub + q < cu1) cat_load<1>(aq[q], va, d, p, d.unit[ub + q], rw, t4);
        }
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          if (ub + q >= cu1) break;
          const CatUnit u = d.unit[ub + q];
          if (u.term < 0) continue;
          uint32_t (&a)[1][4] = aq[q];
          const int rs = d.term[u.term].rs;
          const uint32_t wb = sbase + (uint32_t)((u.woff + ((lq >> 1) * 8 + lr) * rs + (lq & 1) * 8) * 2);
          const uint32_t wb2 = sbase + (uint32_t)((u.woff + lr * rs + (lq & 1) * 8) * 2);
#pragma unroll
          for (int nt = 0; nt < 8; nt += 2) {
            if (nt >= u.nt0 && nt < u.nt1) {
              const uint32_t roff = (uint32_t)(((nt - u.nt0) * 8 * rs) * 2);
              if (nt + 1 < u.nt1) {
                uint32_t b0, b1, b2, b3;
                ldsm_x4(wb + roff, b0, b1, b2, b3);
                mma16816(D[nt], a[0], b0, b1);
                mma16816(D[nt + 1], a[0], b2, b3);
              } else {
                uint32_t b0, b1;
                ldsm_x2(wb2 + roff, b0, b1);
                mma16816(D[nt], a[0], b0, b1);
              }
            } else if (nt + 1 >= u.nt0 && nt + 1 < u.nt1) {
              uint32_t b0, b1;
              ldsm_x2(wb2 + (uint32_t)(((nt + 1 - u.nt0) * 8 * rs) * 2), b0, b1);
              mma16816(D[nt + 1], a[0], b0, b1);
            }
          }
        }
        }
        if (d.relu) {
#pragma unroll
          for (int nt = 0; nt < 8; ++nt)
#pragma unroll
            for (int i = 0; i < 4; ++i) D[nt][i] = fmaxf(D[nt][i], 0.f);
        }
#pragma unroll
        for (int kp = 0; kp < 2; ++kp) {
          uint32_t pa[2][4];
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int ks = 2 * kp + h;
            pa[h][0] = pk2(D[2 * ks][0], D[2 * ks][1]);
            pa[h][1] = pk2(D[2 * ks][2], D[2 * ks][3]);
            pa[h][2] = pk2(D[2 * ks + 1][0], D[2 * ks + 1][1]);
            pa[h][3] = pk2(D[2 * ks + 1][2], D[2 * ks + 1][3]);
          }
#pragma unroll
          for (int nb = 0; nb < NO; ++nb) {
            if (nb >= d.NO) break;
            uint32_t f0, f1, f2, f3;
            ldsm_x4(sbase + (uint32_t)((d.f + (nb * 8 + lr) * d.fs + ch * 64 + kp * 32 + lq * 8) * 2), f0, f1, f2,
                    f3);
            mma16816(O[nb], pa[0], f0, f1);
            mma16816(O[nb], pa[1], f2, f3);
          }
        }
      }
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        if (!rw.ok[h]) continue;
        const int64_t m = ((int64_t)n * d.H + oh) * d.W + rw.wo[h];
#pragma unroll
        for (int nb = 0; nb < NO; ++nb) {
          if (nb >= d.NO) break;
          int k = 0;   // output holding n-tile nb (a merged group's fconvs, reading R37)
          while (k + 1 < d.n_out && nb * 8 >= d.ycol[k + 1]) ++k;
          __nv_bfloat16* yk = reinterpret_cast<__nv_bfloat16*>(p.arena + d.ys[k].off);
          *reinterpret_cast<uint32_t*>(yk + m * (d.ycol[k + 1] - d.ycol[k]) + (nb * 8 - d.ycol[k]) + 2 * t4) =
              pk2(O[nb][2 * h], O[nb][2 * h + 1]);
        }
      }
    }
    __syncthreads();   // the footprint buffer is rewritten by the next tile
  }
}

template <int NO, int PK, int PS, int PP>
void launch_poolcat_t(const CatDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  static bool configured = false;
  static int sms = 148;
  const int PR = (kPcTH - 1) * PS + PK, PC = (kPcTW - 1) * PS + PK;
  const int smem = (d.blob_bytes + 15) / 16 * 16 + PR * PC * kPcStride * 4;
  if (!configured) {
    cudaFuncSetAttribute(mma_poolcat_kernel<NO, PK, PS, PP>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    configured = true;
  }
  int per_sm = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, mma_poolcat_kernel<NO, PK, PS, PP>, 32 * kPcWarps, smem);
  const int tw = (d.W + kPcTW - 1) / kPcTW, th = (d.H + kPcTH - 1) / kPcTH;
  const int ntiles = d.npix / (d.H * d.W) * tw * th;
  const int grid = std::min(ntiles, sms * std::max(per_sm, 1));
  launch_pdl(mma_poolcat_kernel<NO, PK, PS, PP>, dim3(grid), dim3(32 * kPcWarps), smem, s, d, p, tcw, tw, th);
}

// ---------------------------------------------------------------------------
// Chunk-parallel concat kernel for single-level concat groups without a pooled
// member on few pixels (DenseNet-121 blocks 2-4: 25k-100k pixels, C up to 1024 in
// 64-channel chunks of one or two lconv terms each).  The per-block work of the
// generic concat kernel is a long serial chain of (term, tap) units; here each
// warp owns ONE (16-pixel block, 64-channel chunk) pair -- its units' loads all
// in flight together, restore, ReLU, and the chunk's partial reduce GEMM -- and
// the CTA sums the chunks' partial outputs through SMEM (fixed order:
// deterministic, batch-invariant).
// ---------------------------------------------------------------------------
constexpr int kCpWarps = 16;

template <int NO, int KSM>
__global__ void __launch_bounds__(32 * kCpWarps, 1) mma_catp_kernel(const __grid_constant__ CatDesc d, RunPtrs p,
                                                                    const uint16_t* __restrict__ tcw) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int g = lane / 4, t4 = lane % 4;
  {
    const uint4* src = reinterpret_cast<const uint4*>(tcw + d.blob);
    uint4* dst = reinterpret_cast<uint4*>(smem);
    for (int i = threadIdx.x; i < d.blob_bytes / 16; i += blockDim.x) dst[i] = __ldg(src + i);
  }
  __syncthreads();
  pdl_wait();
  pdl_trigger_early();
  const __nv_bfloat16* blob = reinterpret_cast<const __nv_bfloat16*>(smem);
  const float* fb = reinterpret_cast<const float*>(smem + (size_t)d.blob_bf16 * 2);
  float* red = reinterpret_cast<float*>(smem + (d.blob_bytes + 15) / 16 * 16);   // [warp][16][Nout]
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.arena + d.y.off);
  const int lq = lane >> 3, lr = lane & 7;
  const uint32_t sbase = s_u32(blob);
  const int nch = d.nchunks, bpi = kCpWarps / nch;    // blocks per iteration
  const int wb = warp / nch, ch = warp - wb * nch;
  const bool active = wb < bpi;
  const int u0 = d.chunk_u0[ch], u1 = d.chunk_u0[ch + 1];
  for (int it = blockIdx.x; it * bpi < d.nblocks; it += gridDim.x) {
    const int blk = it * bpi + wb;
    if (active && blk < d.nblocks) {
      const CatRows rw = cat_rows(d, blk, g);
      float D[8][4];
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) {
        const float2 b = *reinterpret_cast<const float2*>(fb + d.lbias + ch * 64 + nt * 8 + 2 * t4);
        D[nt][0] = b.x; D[nt][1] = b.y; D[nt][2] = b.x; D[nt][3] = b.y;
      }
      // units in batches of 4: their loads in flight together
      for (int ub = u0; ub < u1; ub += 4) {
        uint32_t a[4][KSM][4];
        bool va[2];
#pragma unroll
        for (int q = 0; q < 4; ++q)
          if (ub + q < u1) cat_load<KSM>(a[q], va, d, p, d.unit[ub + q], rw, t4);
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          if (ub + q >= u1) break;
          const CatUnit u = d.unit[ub + q];
          if (u.term < 0) continue;
          const int nks = d.term[u.term].ks, rs = d.term[u.term].rs;
          const uint32_t wb4 = sbase + (uint32_t)((u.woff + ((lq >> 1) * 8 + lr) * rs + (lq & 1) * 8) * 2);
          const uint32_t wb2 = sbase + (uint32_t)((u.woff + lr * rs + (lq & 1) * 8) * 2);
#pragma unroll
          for (int ks = 0; ks < KSM; ++ks) {
            if (ks >= nks) break;
#pragma unroll
            for (int nt = 0; nt < 8; nt += 2) {
              if (nt >= u.nt0 && nt < u.nt1) {
                const uint32_t roff = (uint32_t)(((nt - u.nt0) * 8 * rs + ks * 16) * 2);
                if (nt + 1 < u.nt1) {
                  uint32_t b0, b1, b2, b3;
                  ldsm_x4(wb4 + roff, b0, b1, b2, b3);
                  mma16816(D[nt], a[q][ks], b0, b1);
                  mma16816(D[nt + 1], a[q][ks], b2, b3);
                } else {
                  uint32_t b0, b1;
                  ldsm_x2(wb2 + roff, b0, b1);
                  mma16816(D[nt], a[q][ks], b0, b1);
                }
              } else if (nt + 1 >= u.nt0 && nt + 1 < u.nt1) {
                uint32_t b0, b1;
                ldsm_x2(wb2 + (uint32_t)(((nt + 1 - u.nt0) * 8 * rs + ks * 16) * 2), b0, b1);
                mma16816(D[nt + 1], a[q][ks], b0, b1);
              }
            }
          }
        }
      }
      if (d.relu) {
#pragma unroll
        for (int nt = 0; nt < 8; ++nt)
#pragma unroll
          for (int i = 0; i < 4; ++i) D[nt][i] = fmaxf(D[nt][i], 0.f);
      }
      float O[NO][4];
#pragma unroll
      for (int i = 0; i < NO; ++i) O[i][0] = O[i][1] = O[i][2] = O[i][3] = 0.f;
#pragma unroll
      for (int kp = 0; kp < 2; ++kp) {
        uint32_t pa[2][4];
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int ks = 2 * kp + h;
          pa[h][0] = pk2(D[2 * ks][0], D[2 * ks][1]);
          pa[h][1] = pk2(D[2 * ks][2], D[2 * ks][3]);
          pa[h][2] = pk2(D[2 * ks + 1][0], D[2 * ks + 1][1]);
          pa[h][3] = pk2(D[2 * ks + 1][2], D[2 * ks + 1][3]);
        }
#pragma unroll
        for (int nb = 0; nb < NO; ++nb) {
          if (nb >= d.NO) break;
          uint32_t f0, f1, f2, f3;
          ldsm_x4(sbase + (uint32_t)((d.f + (nb * 8 + lr) * d.fs + ch * 64 + kp * 32 + lq * 8) * 2), f0, f1, f2, f3);
          mma16816(O[nb], pa[0], f0, f1);
          mma16816(O[nb], pa[1], f2, f3);
        }
      }
      float* rwp = red + (size_t)warp * 16 * d.Nout;
#pragma unroll
      for (int nb = 0; nb < NO; ++nb) {
        if (nb >= d.NO) break;
        const int col = nb * 8 + 2 * t4;
        *reinterpret_cast<float2*>(rwp + g * d.Nout + col) = make_float2(O[nb][0], O[nb][1]);
        *reinterpret_cast<float2*>(rwp + (g + 8) * d.Nout + col) = make_float2(O[nb][2], O[nb][3]);
      }
    }
    __syncthreads();
    // sum the chunks' partials (chunk order fixed) and store bf16 pairs
    const int per_blk = 16 * d.Nout / 2;
    for (int i = threadIdx.x; i < bpi * per_blk; i += blockDim.x) {
      const int b = i / per_blk, e = (i - b * per_blk) * 2;
      const int blk = it * bpi + b;
      const int m = blk * 16 + e / d.Nout;
      if (blk >= d.nblocks || m >= d.npix) continue;
      float s0 = 0.f, s1 = 0.f;
      for (int c = 0; c < nch; ++c) {
        const float2 v = *reinterpret_cast<const float2*>(red + (size_t)(b * nch + c) * 16 * d.Nout + e);
        s0 += v.x;
        s1 += v.y;
      }
      *reinterpret_cast<uint32_t*>(y + (int64_t)m * d.Nout + e % d.Nout) = pk2(s0, s1);
    }
    __syncthreads();
  }
}

template <int NO, int KSM>
void launch_catp_t(const CatDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  static bool configured = false;
  static int sms = 148;
  const int smem = (d.blob_bytes + 15) / 16 * 16 + kCpWarps * 16 * d.Nout * 4;
  if (!configured) {
    cudaFuncSetAttribute(mma_catp_kernel<NO, KSM>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    configured = true;
  }
  const int bpi = kCpWarps / d.nchunks;
  const int grid = std::min((d.nblocks + bpi - 1) / bpi, sms);
  launch_pdl(mma_catp_kernel<NO, KSM>, dim3(grid), dim3(32 * kCpWarps), smem, s, d, p, tcw);
}

template <int KSM, bool POOL>
void launch_cat_no(const CatDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  switch ((d.NO + 1) / 2) {
    case 1: return launch_cat_t<2, KSM, POOL>(d, tcw, p, s);
    case 2: return launch_cat_t<4, KSM, POOL>(d, tcw, p, s);
    case 3: return launch_cat_t<6, KSM, POOL>(d, tcw, p, s);
    default: return launch_cat_t<8, KSM, POOL>(d, tcw, p, s);
  }
}

}  // namespace

bool mma_catp_ok(const CatDesc& d) {
  // measured (B200): wins only where the tcgen05 kernel's 128-pixel tiles leave most SMs idle
  // (ResNet-18c stages 3-4: 16-64 tiles); 1.5-2x slower than tcgen05 on DenseNet's blocks 2-4
  if (d.pool != 0 || d.nchunks > 8 || d.npix >= 74 * 128 || d.n_out > 1) return false;
  for (int j = 0; j < d.n_terms; ++j)
    if (d.term[j].ks > 4) return false;
  return (d.blob_bytes + 15) / 16 * 16 + kCpWarps * 16 * d.Nout * 4 <= 227 * 1024;
}

bool mma_poolcat_ok(const CatDesc& d) {
  const bool win = (d.pk == 3 && d.ps == 2 && d.pp == 1) || (d.pk == 2 && d.ps == 2 && d.pp == 0);
  if (d.pool != 1 || !win || d.pc0 != 0 || d.pc1 != 1 || d.NO > 6) return false;
  if (d.n_terms != d.n_plain + 1 || d.term[d.n_plain].R > 16) return false;
  for (int j = 0; j < d.n_plain; ++j)
    if (d.term[j].tk != 1 || d.term[j].R > 16) return false;
  const int PR = (kPcTH - 1) * d.ps + d.pk, PC = (kPcTW - 1) * d.ps + d.pk;
  return (d.blob_bytes + 15) / 16 * 16 + PR * PC * kPcStride * 4 <= 227 * 1024;
}

void launch_mma_cat(const CatDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  if (mma_catp_ok(d)) {
    int ksm = 1;
    for (int j = 0; j < d.n_terms; ++j) ksm = std::max(ksm, d.term[j].ks);
    const int no2 = (d.NO + 1) / 2;
#define TEMCO_CATP(n, k) if ((no2 * 2 <= n) && ksm <= k) return launch_catp_t<n, k>(d, tcw, p, s);
    TEMCO_CATP(2, 1) TEMCO_CATP(2, 2) TEMCO_CATP(2, 4) TEMCO_CATP(4, 1) TEMCO_CATP(4, 2) TEMCO_CATP(4, 4)
    TEMCO_CATP(8, 1) TEMCO_CATP(8, 2) TEMCO_CATP(8, 4)
#undef TEMCO_CATP
  }
  if (mma_poolcat_ok(d)) {
    if (d.pk == 2) {   // VGG's 2x2 / stride-2 pools
      if (d.NO == 1) return launch_poolcat_t<1, 2, 2, 0>(d, tcw, p, s);
      if (d.NO == 2) return launch_poolcat_t<2, 2, 2, 0>(d, tcw, p, s);
      if (d.NO <= 4) return launch_poolcat_t<4, 2, 2, 0>(d, tcw, p, s);
      return launch_poolcat_t<6, 2, 2, 0>(d, tcw, p, s);
    }
    if (d.NO == 1) return launch_poolcat_t<1, 3, 2, 1>(d, tcw, p, s);
    if (d.NO == 2) return launch_poolcat_t<2, 3, 2, 1>(d, tcw, p, s);
    if (d.NO <= 4) return launch_poolcat_t<4, 3, 2, 1>(d, tcw, p, s);   // 3 or 4 n-tiles (bounded by d.NO inside)
    return launch_poolcat_t<6, 3, 2, 1>(d, tcw, p, s);   // a merged group's stacked F (R37): 5 or 6 n-tiles
  }
  int ksm = 1;
  for (int j = 0; j < d.n_terms; ++j) ksm = std::max(ksm, d.term[j].ks);
  const bool pool = d.pool != 0;
  if (ksm == 1) return pool ? launch_cat_no<1, true>(d, tcw, p, s) : launch_cat_no<1, false>(d, tcw, p, s);
  if (ksm == 2) return pool ? launch_cat_no<2, true>(d, tcw, p, s) : launch_cat_no<2, false>(d, tcw, p, s);
  return pool ? launch_cat_no<4, true>(d, tcw, p, s) : launch_cat_no<4, false>(d, tcw, p, s);
}

}  // namespace temco
