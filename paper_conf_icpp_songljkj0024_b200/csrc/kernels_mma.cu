// Register-resident fused restore -> BN -> add -> ReLU -> [pool] -> reduce
// kernel with mma.sync m16n8k16 (see mma_chain.h).
//
// Each warp owns 16 output pixels at a time.  Its reduced inputs are staged in
// a per-warp SMEM double buffer with 16-byte cp.async (the next block / tap is
// in flight while the current one computes), all weights (BN-folded Lhat,
// F, level biases) are SMEM-resident for the whole persistent CTA.  For a
// restored chunk of CH channels the accumulator fragments D[CH/8][4] hold the
// 16 x CH restored tile in registers; bias / ReLU / max-pool run on them; then
// they are re-packed to bf16 as the A operand of the reduce GEMM (the fp32
// m16n8k16 C layout equals the bf16 A layout pairwise), accumulating out[16 x
// Nout] in registers across chunks.  The C-wide tensor never leaves registers.
#include <cuda_bf16.h>

#include <algorithm>
#include <cmath>

#include "chain_parse.h"
#include "mma_chain.h"

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

bool mma_lower_chain(const IR& ir, const Step& s, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                     MmaChainDesc& d) {
  const Node& root = ir.nodes[s.out];
  if (root.role != ROLE_FCONV) return false;
  const int tsrc = ir.oin[s.out][0];
  const Node& tn = ir.nodes[tsrc];
  const int C = tn.C, Nout = root.C;
  if (Nout % 8 || Nout > 128 || C % 16) return false;
  int pool = 0, pk = 1, ps = 1, pp = 0, csrc = tsrc;
  if ((tn.op == OP_MAXPOOL || tn.op == OP_AVGPOOL) && s.members.size() > 2) {
    pool = tn.op == OP_MAXPOOL ? 1 : 2;
    pk = tn.kh; ps = tn.sh; pp = tn.ph;
    csrc = ir.oin[tsrc][0];
  }
  const Node& cn = ir.nodes[csrc];
  ChainParser P{ir, std::set<int>(s.members.begin(), s.members.end()), C, {}, cn.H, cn.W};
  P.allow_silu = true;   // act_apply: 1 ReLU, 2 SiLU
  P.members.erase(s.out);
  if (pool) P.members.erase(tsrc);
  std::vector<PLevel> levels;
  if (!P.chain(csrc, levels)) return false;
  if (P.visited != P.members) return false;
  int nterms = 0;
  for (auto& L : levels) {
    nterms += (int)L.terms.size();
    if (!L.pm.empty()) return false;                 // pooled concat members: tcgen05 / generic paths
    for (auto& t : L.terms)
      if (t.tk > 1) return false;
  }
  if ((int)levels.size() > kMmaMaxLevels || nterms > kMmaMaxTerms) return false;
  for (auto& L : levels)
    for (auto& t : L.terms) {
      const int r = ir.oin[t.lconv][0];
      const Loc& l = loc.at(r);
      if (l.where != W_ARENA || l.dtype != DT_BF16 || ir.nodes[r].C % 8 || ir.nodes[t.lconv].C % 8) return false;
    }
  const Loc& yl = loc.at(s.out);
  if (yl.where != W_ARENA || yl.dtype != DT_BF16) return false;

  d = MmaChainDesc();
  d.C = C;
  d.CH = C <= 64 ? 64 : 128;
  d.Cpad = (C + d.CH - 1) / d.CH * d.CH;
  d.nchunks = d.Cpad / d.CH;
  d.Nout = Nout;
  d.Np8 = Nout;
  d.pool = pool; d.pk = pk; d.ps = ps; d.pp = pp; d.taps = pk * pk;
  d.Hin = cn.H; d.Win = cn.W; d.Ho = tn.H; d.Wo = tn.W;
  d.npix = (int64_t)ir.batch * tn.H * tn.W;
  d.nblocks = (int)((d.npix + 15) / 16);
  d.y = yl;
  d.n_levels = (int)levels.size();
  // blob: [Lhat_j rows (Rp + 8)] ... [F (Cpad + 8)] | fp32 biases
  std::vector<uint16_t> blob;
  std::vector<float> biases;
  int j = 0, astride = 0;
  int64_t fl_terms = 0, by_terms = 0;
  for (int l = 0; l < d.n_levels; ++l) {
    const PLevel& L = levels[l];
    d.relu[l] = L.relu ? 1 : L.silu ? 2 : 0;
    d.bias[l] = (int32_t)biases.size();
    for (int c = 0; c < d.Cpad; ++c) biases.push_back(c < C ? (float)L.bias[c] : 0.f);
    for (const PTerm& t : L.terms) {
      const Node& lc = ir.nodes[t.lconv];
      const int r = ir.oin[t.lconv][0];
      const int R = ir.nodes[r].C;
      MmaTerm& T = d.term[j++];
      T.r = loc.at(r);
      T.R = R;
      T.Rp = (R + 15) / 16 * 16;
      T.c0 = t.c0;
      T.C = lc.C;
      T.level = l;
      T.w = (int32_t)blob.size();
      const int rs = T.Rp + 8;
      blob.resize(blob.size() + (size_t)lc.C * rs, 0);
      for (int c = 0; c < lc.C; ++c)
        for (int k = 0; k < R; ++k)
          blob[T.w + (size_t)c * rs + k] = f2bf((float)(t.scale[c] * (*lc.w)[(size_t)c * R + k]));
      astride += rs;
      fl_terms += 2LL * lc.C * R;
      by_terms += 2LL * R;
    }
    d.lvl_end[l] = j;
  }
  d.n_terms = j;
  if (((astride / 8) & 1) == 0) astride += 8;   // odd number of 16-byte chunks per row: conflict-free ldmatrix
  d.a_stride = astride;
  d.f = (int32_t)blob.size();
  const int fs = d.Cpad + 8;
  blob.resize(blob.size() + (size_t)d.Np8 * fs, 0);
  for (int o = 0; o < Nout; ++o)
    for (int c = 0; c < C; ++c) blob[d.f + (size_t)o * fs + c] = f2bf((*root.w)[(size_t)o * C + c]);
  if (root.b) return false;                      // fconv factors carry no bias (O1)
  while (blob.size() % 8) blob.push_back(0);
  d.blob_bf16 = (int32_t)blob.size();
  for (float b : biases) {
    uint32_t u;
    memcpy(&u, &b, 4);
    blob.push_back((uint16_t)(u & 0xFFFF));
    blob.push_back((uint16_t)(u >> 16));
  }
  while (blob.size() % 8) blob.push_back(0);
  d.blob_bytes = (int32_t)blob.size() * 2;
  // per-warp prefetch ring: as deep as 8 units within ~200 KB (16 warps for
  // 64-wide chunks, 8 for 128-wide ones, whose fragments need > 128 registers)
  const int unit_bytes = 16 * d.a_stride * 2;
  d.warps = d.CH == 64 ? 16 : 8;
  d.nbuf = std::min(8, (200 * 1024 - d.blob_bytes - 256) / (d.warps * unit_bytes));
  if (d.nbuf < 2) return false;
  d.smem_bytes = d.blob_bytes + d.warps * d.nbuf * unit_bytes + 256;
  while (tcw.size() % 512) tcw.push_back(0);
  d.blob = (int64_t)tcw.size();
  tcw.insert(tcw.end(), blob.begin(), blob.end());
  const int64_t nin = (int64_t)ir.batch * cn.H * cn.W;
  d.alg_flops = nin * fl_terms + d.npix * 2LL * Nout * C;
  d.alg_bytes = nin * by_terms + d.npix * 2LL * Nout;
  // the generic kernel keeps a pooled chain's running max in registers (one
  // 64-wide chunk); the lean kernel walks chunks as units
  if (pool && C > 64 && !mma_lean_ok(d)) return false;
  return true;
}

namespace {

// level activation: 1 ReLU, 2 SiLU (h + h tanh(h), h = x / 2, one tanh.approx: bf16 outputs)
__device__ __forceinline__ float act_apply(float x, int act) {
  if (act == 2) {
    const float h = 0.5f * x;
    float t;
    asm("tanh.approx.f32 %0, %1;" : "=f"(t) : "f"(h));
    return fmaf(h, t, h);
  }
  return fmaxf(x, 0.f);
}

__device__ __forceinline__ uint32_t s_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void ldsm_x4(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0, %1, %2, %3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}

__device__ __forceinline__ void ldsm_x2(uint32_t addr, uint32_t& r0, uint32_t& r1) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x2.shared.b16 {%0, %1}, [%2];" : "=r"(r0), "=r"(r1) : "r"(addr));
}

__device__ __forceinline__ void mma16816(float (&c)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                         uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0, %1, %2, %3}, {%4, %5, %6, %7}, {%8, %9}, "
      "{%0, %1, %2, %3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

__device__ __forceinline__ void cp16(uint32_t dst, const void* src, uint32_t bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(bytes) : "memory");
}

__device__ __forceinline__ uint32_t pk2(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}


// cp.async.wait_group takes an immediate: dispatch the ring depth
__device__ __forceinline__ void cp_async_wait_dyn(int n) {
  switch (n) {
    case 1: asm volatile("cp.async.wait_group 1;" ::: "memory"); break;
    case 2: asm volatile("cp.async.wait_group 2;" ::: "memory"); break;
    case 3: asm volatile("cp.async.wait_group 3;" ::: "memory"); break;
    case 4: asm volatile("cp.async.wait_group 4;" ::: "memory"); break;
    case 5: asm volatile("cp.async.wait_group 5;" ::: "memory"); break;
    case 6: asm volatile("cp.async.wait_group 6;" ::: "memory"); break;
    default: asm volatile("cp.async.wait_group 7;" ::: "memory"); break;
  }
}

// stage the A rows of unit u (a 16-pixel block, and for a pooled chain one tap)
__device__ __forceinline__ void stage_unit(const MmaChainDesc& d, const RunPtrs& p, __nv_bfloat16* st, int64_t blk,
                                           int tap, int lane) {
  int off = 0;
  for (int j = 0; j < d.n_terms; ++j) {
    const MmaTerm& t = d.term[j];
    const uint8_t* rb = reinterpret_cast<const uint8_t*>(p.arena + t.r.off);
    const int cpr = t.Rp / 8;                     // 16-byte chunks per row (incl. K padding)
    for (int c = lane; c < 16 * cpr; c += 32) {
      const int row = c / cpr, q = c - row * cpr;
      const int64_t m = blk * 16 + row;
      int64_t pix = m;
      bool ok = m < d.npix && q * 8 < t.R;
      if (d.pool && ok) {
        const int hw = d.Ho * d.Wo;
        const int n = (int)(m / hw), rem = (int)(m % hw);
        const int hi = (rem / d.Wo) * d.ps - d.pp + tap / d.pk, wi = (rem % d.Wo) * d.ps - d.pp + tap % d.pk;
        ok = hi >= 0 && hi < d.Hin && wi >= 0 && wi < d.Win;
        pix = ((int64_t)n * d.Hin + hi) * d.Win + wi;
      }
      cp16(s_u32(st + row * d.a_stride + off + q * 8), ok ? rb + (pix * t.R + q * 8) * 2 : rb, ok ? 16u : 0u);
    }
    off += t.Rp + 8;
  }
}

template <int CH, int NO, bool POOL, int kWarps>
__global__ void __launch_bounds__(32 * kWarps, 1) mma_chain_kernel(const __grid_constant__ MmaChainDesc d, RunPtrs p,
                                                                   const uint16_t* __restrict__ tcw) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int g = lane / 4, t4 = lane % 4;
  // weights -> SMEM (once per persistent CTA)
  {
    const uint4* src = reinterpret_cast<const uint4*>(tcw + d.blob);
    uint4* dst = reinterpret_cast<uint4*>(smem);
    for (int i = threadIdx.x; i < d.blob_bytes / 16; i += blockDim.x) dst[i] = __ldg(src + i);
  }
  __syncthreads();
  const __nv_bfloat16* blob = reinterpret_cast<const __nv_bfloat16*>(smem);
  const float* fb = reinterpret_cast<const float*>(smem + (size_t)d.blob_bf16 * 2);
  __nv_bfloat16* stage = reinterpret_cast<__nv_bfloat16*>(smem + d.blob_bytes) + (size_t)warp * d.nbuf * 16 * d.a_stride;
  const int units_per_blk = POOL ? d.taps : 1;
  const int64_t gw = (int64_t)blockIdx.x * kWarps + warp, nw = (int64_t)gridDim.x * kWarps;
  // ldmatrix lane addressing (A: 16 rows x 16 k; B: 8 rows x 16 k)
  const int a_row = (lane & 7) + ((lane >> 3) & 1) * 8, a_col = (lane >> 4) * 8;
  const int b_row = lane & 7, b_col = ((lane >> 3) & 1) * 8;

  // NB-deep per-warp prefetch ring over the warp's unit sequence (block, tap):
  // these groups are HBM-bound with a few hundred bytes per unit, so many units
  // must be in flight per warp to cover the memory latency (Little's law)
  const int NB = d.nbuf;
  const int ustride = 16 * d.a_stride;
  int64_t pblk = gw;
  int ptap = 0;
  auto advance = [&](int64_t& b, int& t) {
    if (++t == units_per_blk) t = 0, b += nw;
  };
  for (int k = 0; k < NB - 1; ++k) {
    if (pblk < d.nblocks) stage_unit(d, p, stage + k * ustride, pblk, ptap, lane);
    asm volatile("cp.async.commit_group;" ::: "memory");
    advance(pblk, ptap);
  }
  int64_t blk = gw;
  int tap = 0;
  int buf = 0, pbuf = NB - 1;

  float O[NO][4];
  float run[POOL ? CH / 8 : 1][4];
  while (blk < d.nblocks) {
    if (pblk < d.nblocks) stage_unit(d, p, stage + pbuf * ustride, pblk, ptap, lane);
    asm volatile("cp.async.commit_group;" ::: "memory");
    advance(pblk, ptap);
    if (++pbuf == NB) pbuf = 0;
    cp_async_wait_dyn(NB - 1);
    __syncwarp();
    const __nv_bfloat16* A = stage + buf * ustride;
    int64_t nblk = blk;
    int ntap = tap;
    advance(nblk, ntap);

    if (tap == 0) {
#pragma unroll
      for (int i = 0; i < NO; ++i) O[i][0] = O[i][1] = O[i][2] = O[i][3] = 0.f;
    }
    // validity of rows g, g+8 for this tap (pooled chains)
    bool v0 = true, v1 = true;
    if (POOL) {
      const int hw = d.Ho * d.Wo;
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int64_t m = blk * 16 + g + 8 * h;
        const int rem = (int)(m % hw);
        const int hi = (rem / d.Wo) * d.ps - d.pp + tap / d.pk, wi = (rem % d.Wo) * d.ps - d.pp + tap % d.pk;
        const bool v = hi >= 0 && hi < d.Hin && wi >= 0 && wi < d.Win;
        (h ? v1 : v0) = v;
      }
    }
    for (int ch = 0; ch < d.nchunks; ++ch) {
      float D[CH / 8][4];
      int toff = 0, j = 0;
      for (int l = 0; l < d.n_levels; ++l) {
        const float* bl = fb + d.bias[l] + ch * CH;
#pragma unroll
        for (int nb = 0; nb < CH / 8; ++nb) {
          const float b0 = bl[nb * 8 + 2 * t4], b1 = bl[nb * 8 + 2 * t4 + 1];
          if (l == 0) {
            D[nb][0] = b0; D[nb][1] = b1; D[nb][2] = b0; D[nb][3] = b1;
          } else {
            D[nb][0] += b0; D[nb][1] += b1; D[nb][2] += b0; D[nb][3] += b1;
          }
        }
        for (; j < d.lvl_end[l]; ++j) {
          const MmaTerm& T = d.term[j];
          const int lo = T.c0 - ch * CH, hi = lo + T.C;     // term's columns relative to the chunk
          if (hi > 0 && lo < CH) {
            const int rs = T.Rp + 8;
            for (int ks = 0; ks < T.Rp / 16; ++ks) {
              uint32_t a0, a1, a2, a3;
              ldsm_x4(s_u32(A + a_row * d.a_stride + toff + ks * 16 + a_col), a0, a1, a2, a3);
#pragma unroll
              for (int nb = 0; nb < CH / 8; ++nb) {
                if (nb * 8 >= lo && nb * 8 < hi) {
                  uint32_t b0, b1;
                  ldsm_x2(s_u32(blob + T.w + (nb * 8 - lo + b_row) * rs + ks * 16 + b_col), b0, b1);
                  mma16816(D[nb], a0, a1, a2, a3, b0, b1);
                }
              }
            }
          }
          toff += T.Rp + 8;
        }
        if (d.relu[l]) {
#pragma unroll
          for (int nb = 0; nb < CH / 8; ++nb)
#pragma unroll
            for (int i = 0; i < 4; ++i) D[nb][i] = act_apply(D[nb][i], d.relu[l]);
        }
      }
      if (POOL) {
        // running max / sum over taps (CH == C: single chunk)
#pragma unroll
        for (int nb = 0; nb < CH / 8; ++nb) {
          if (d.pool == 1) {
            const float n0 = v0 ? 0.f : -INFINITY, n1 = v1 ? 0.f : -INFINITY;
            const float x0 = D[nb][0] + n0, x1 = D[nb][1] + n0, x2 = D[nb][2] + n1, x3 = D[nb][3] + n1;
            if (tap == 0) {
              run[nb][0] = x0; run[nb][1] = x1; run[nb][2] = x2; run[nb][3] = x3;
            } else {
              run[nb][0] = fmaxf(run[nb][0], x0); run[nb][1] = fmaxf(run[nb][1], x1);
              run[nb][2] = fmaxf(run[nb][2], x2); run[nb][3] = fmaxf(run[nb][3], x3);
            }
          } else {
#pragma unroll
            for (int i = 0; i < 4; ++i) run[nb][i] = tap == 0 ? D[nb][i] : run[nb][i] + D[nb][i];
          }
        }
        if (tap != d.taps - 1) continue;
        const float sc = d.pool == 2 ? 1.f / (float)d.taps : 1.f;
#pragma unroll
        for (int nb = 0; nb < CH / 8; ++nb)
#pragma unroll
          for (int i = 0; i < 4; ++i) D[nb][i] = run[nb][i] * sc;
      }
      // reduce: out[16 x Nout] += P[16 x CH] F[:, chunk]^T, P re-packed from D
      const int fs = d.Cpad + 8;
#pragma unroll
      for (int ks = 0; ks < CH / 16; ++ks) {
        const uint32_t a0 = pk2(D[2 * ks][0], D[2 * ks][1]), a1 = pk2(D[2 * ks][2], D[2 * ks][3]);
        const uint32_t a2 = pk2(D[2 * ks + 1][0], D[2 * ks + 1][1]), a3 = pk2(D[2 * ks + 1][2], D[2 * ks + 1][3]);
#pragma unroll
        for (int nb = 0; nb < NO; ++nb) {
          if (nb * 8 < d.Nout) {
            uint32_t b0, b1;
            ldsm_x2(s_u32(blob + d.f + (nb * 8 + b_row) * fs + ch * CH + ks * 16 + b_col), b0, b1);
            mma16816(O[nb], a0, a1, a2, a3, b0, b1);
          }
        }
      }
    }
    if (!POOL || tap == d.taps - 1) {
      __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.arena + d.y.off);
      const int64_t m0 = blk * 16 + g, m1 = m0 + 8;
#pragma unroll
      for (int nb = 0; nb < NO; ++nb) {
        if (nb * 8 < d.Nout) {
          const int col = nb * 8 + 2 * t4;
          if (m0 < d.npix) *reinterpret_cast<uint32_t*>(y + m0 * d.Nout + col) = pk2(O[nb][0], O[nb][1]);
          if (m1 < d.npix) *reinterpret_cast<uint32_t*>(y + m1 * d.Nout + col) = pk2(O[nb][2], O[nb][3]);
        }
      }
    }
    __syncwarp();
    if (++buf == NB) buf = 0;
    tap = ntap;
    blk = nblk;
  }
  asm volatile("cp.async.wait_group 0;" ::: "memory");
}

template <int CH, int NO, bool POOL>
void launch_t(const MmaChainDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  static bool configured = false;
  static int sms = 148;
  if (!configured) {
    cudaFuncSetAttribute(mma_chain_kernel<CH, NO, POOL, (CH == 64 ? 16 : 8)>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    configured = true;
  }
  const int per_sm = 1;   // 16 warps x ~100 registers: one persistent CTA per SM
  const int grid = (int)std::min<int64_t>((d.nblocks + d.warps - 1) / d.warps, (int64_t)sms * per_sm);
  mma_chain_kernel<CH, NO, POOL, (CH == 64 ? 16 : 8)><<<grid, 32 * d.warps, d.smem_bytes, s>>>(d, p, tcw);
}


// ---------------------------------------------------------------------------
// Lean variant for the commonest HBM-bound shape: one level, one reduced input
// (lconv -> BN -> [ReLU] -> fconv; VGG's per-conv groups, ResNet's in-block
// groups), rank <= 32, C % 64 == 0, Nout <= 32.  Straight-line templated code:
// the A fragments come straight from global memory into registers (two 32-bit
// loads per row pair and k-step; the next block's are in flight while the
// current one computes), the weights are ldmatrix'd from SMEM, the restored
// 16 x 64 chunk lives in 32 accumulator registers and is re-packed in place
// as the A operand of the reduce GEMM.  ~100 instructions per 16 pixels.
// ---------------------------------------------------------------------------
constexpr int kLeanWarps = 16;

// unit = (16-pixel output block, 64-channel chunk, pool tap); a warp walks its
// blocks' units in that order, with the A fragments of the next two units in
// flight.  Pooled groups gather the tap-shifted input rows (zero rows, masked
// to -inf for a max pool, outside the image).
struct LeanCursor {
  int64_t blk;
  int ch, tap;
  int hi0[2], wi0[2], nrow[2];   // pooled: per fragment row, the tap window origin and n * Hin
};

// (re)compute the per-row pool window origins when a cursor enters a new block
__device__ __forceinline__ void lean_set_block(const MmaChainDesc& d, LeanCursor& u, int g) {
  if (!d.pool) return;
  const int hw = d.Ho * d.Wo;
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    const int m = (int)(u.blk * 16) + g + 8 * h;
    const int n = m / hw, rem = m - n * hw;
    const int ho = rem / d.Wo, wo = rem - ho * d.Wo;
    u.hi0[h] = ho * d.ps - d.pp;
    u.wi0[h] = wo * d.ps - d.pp;
    u.nrow[h] = n * d.Hin;
  }
}

template <int KS>
__device__ __forceinline__ void lean_load_a(uint32_t (&a)[KS][4], const MmaChainDesc& d, const uint32_t* __restrict__ r,
                                            const LeanCursor& u, int R, int g, int t4) {
  const int64_t m0 = u.blk * 16 + g, m1 = m0 + 8;
  int64_t p0 = m0, p1 = m1;
  bool v0 = m0 < d.npix, v1 = m1 < d.npix;
  if (d.pool) {
    const int ty = u.tap / d.pk, tx = u.tap - ty * d.pk;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int hi = u.hi0[h] + ty, wi = u.wi0[h] + tx;
      const bool v = (h ? v1 : v0) && hi >= 0 && hi < d.Hin && wi >= 0 && wi < d.Win;
      const int64_t pix = (int64_t)(u.nrow[h] + hi) * d.Win + wi;
      if (h) v1 = v, p1 = pix; else v0 = v, p0 = pix;
    }
  }
  const int rw = R / 2;   // 32-bit words per row
#pragma unroll
  for (int ks = 0; ks < KS; ++ks) {
    const int k0 = ks * 16 + 2 * t4, k1 = k0 + 8;
    a[ks][0] = (v0 && k0 < R) ? __ldg(r + p0 * rw + k0 / 2) : 0u;
    a[ks][1] = (v1 && k0 < R) ? __ldg(r + p1 * rw + k0 / 2) : 0u;
    a[ks][2] = (v0 && k1 < R) ? __ldg(r + p0 * rw + k1 / 2) : 0u;
    a[ks][3] = (v1 && k1 < R) ? __ldg(r + p1 * rw + k1 / 2) : 0u;
  }
}

// is fragment row h's tap inside the image (max-pool masking)
__device__ __forceinline__ bool lean_tap_valid(const MmaChainDesc& d, const LeanCursor& u, int h) {
  const int ty = u.tap / d.pk, tx = u.tap - ty * d.pk;
  const int hi = u.hi0[h] + ty, wi = u.wi0[h] + tx;
  return hi >= 0 && hi < d.Hin && wi >= 0 && wi < d.Win;
}

template <int KS, int NO>
__global__ void __launch_bounds__(32 * kLeanWarps, 1) mma_lean_kernel(const __grid_constant__ MmaChainDesc d,
                                                                      RunPtrs p, const uint16_t* __restrict__ tcw) {
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
  const float* fb = reinterpret_cast<const float*>(smem + (size_t)d.blob_bf16 * 2) + d.bias[0];
  const MmaTerm& T = d.term[0];
  const uint32_t* r = reinterpret_cast<const uint32_t*>(p.arena + T.r.off);
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.arena + d.y.off);
  const int rs = T.Rp + 8, fs = d.Cpad + 8;
  const int relu = d.relu[0];
  const int taps = d.pool ? d.taps : 1;
  const int nch = d.Cpad / 64;
  // ldmatrix.x4 lane addressing: matrix q = lane / 8 -> (n-tile + q / 2, k half q % 2)
  const int lq = lane >> 3, lr = lane & 7;
  const uint32_t wbase = s_u32(blob + T.w + ((lq >> 1) * 8 + lr) * rs + (lq & 1) * 8);
  const uint32_t fbase = s_u32(blob + d.f + lr * fs + lq * 8);
  const int64_t nw = (int64_t)gridDim.x * kLeanWarps;
  auto advance = [&](LeanCursor& u) {
    if (++u.tap == taps) {
      u.tap = 0;
      if (++u.ch == nch) {
        u.ch = 0;
        u.blk += nw;
        if (u.blk < d.nblocks) lean_set_block(d, u, g);
      }
    }
  };
  LeanCursor cur{};
  cur.blk = (int64_t)blockIdx.x * kLeanWarps + warp;
  if (cur.blk < d.nblocks) lean_set_block(d, cur, g);
  LeanCursor pf = cur;
  uint32_t a[KS][4], an[KS][4], ann[KS][4];
  // unpooled groups: a block's later 64-channel chunks read the same A rows -- reuse the
  // fragments of the unit before instead of reloading them
  if (pf.blk < d.nblocks) lean_load_a<KS>(a, d, r, pf, T.R, g, t4);
  advance(pf);
  if (!d.pool && pf.ch > 0) {
#pragma unroll
    for (int ks = 0; ks < KS; ++ks)
#pragma unroll
      for (int i = 0; i < 4; ++i) an[ks][i] = a[ks][i];
  } else if (pf.blk < d.nblocks) {
    lean_load_a<KS>(an, d, r, pf, T.R, g, t4);
  }
  advance(pf);
  float O[NO][4];
  float run[8][4];
  const float sc = d.pool == 2 ? 1.f / (float)d.taps : 1.f;
  for (; cur.blk < d.nblocks; advance(cur)) {
    if (!d.pool && pf.ch > 0) {
#pragma unroll
      for (int ks = 0; ks < KS; ++ks)
#pragma unroll
        for (int i = 0; i < 4; ++i) ann[ks][i] = an[ks][i];
    } else if (pf.blk < d.nblocks) {
      lean_load_a<KS>(ann, d, r, pf, T.R, g, t4);
    }
    advance(pf);
    const int c0 = cur.ch * 64;
    if (cur.ch == 0 && cur.tap == 0) {
#pragma unroll
      for (int i = 0; i < NO; ++i) O[i][0] = O[i][1] = O[i][2] = O[i][3] = 0.f;
    }
    float D[8][4];
#pragma unroll
    for (int nt = 0; nt < 8; ++nt) {
      const float2 b = *reinterpret_cast<const float2*>(fb + c0 + nt * 8 + 2 * t4);
      D[nt][0] = b.x; D[nt][1] = b.y; D[nt][2] = b.x; D[nt][3] = b.y;
    }
#pragma unroll
    for (int ks = 0; ks < KS; ++ks)
#pragma unroll
      for (int np = 0; np < 4; ++np) {
        uint32_t b0, b1, b2, b3;
        ldsm_x4(wbase + (uint32_t)(((c0 + np * 16) * rs + ks * 16) * 2), b0, b1, b2, b3);
        mma16816(D[2 * np], a[ks][0], a[ks][1], a[ks][2], a[ks][3], b0, b1);
        mma16816(D[2 * np + 1], a[ks][0], a[ks][1], a[ks][2], a[ks][3], b2, b3);
      }
    if (relu) {
#pragma unroll
      for (int nt = 0; nt < 8; ++nt)
#pragma unroll
        for (int i = 0; i < 4; ++i) D[nt][i] = act_apply(D[nt][i], relu);
    }
    bool last = true;
    if (d.pool) {
      // fold this tap into the running max / sum (max: taps outside the image excluded)
      float n0 = 0.f, n1 = 0.f;
      if (d.pool == 1) {
        n0 = lean_tap_valid(d, cur, 0) ? 0.f : -INFINITY;
        n1 = lean_tap_valid(d, cur, 1) ? 0.f : -INFINITY;
      }
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) {
        const float x[4] = {D[nt][0] + n0, D[nt][1] + n0, D[nt][2] + n1, D[nt][3] + n1};
#pragma unroll
        for (int i = 0; i < 4; ++i)
          run[nt][i] = cur.tap == 0 ? x[i] : d.pool == 1 ? fmaxf(run[nt][i], x[i]) : run[nt][i] + x[i];
      }
      last = cur.tap == taps - 1;
      if (last) {
#pragma unroll
        for (int nt = 0; nt < 8; ++nt)
#pragma unroll
          for (int i = 0; i < 4; ++i) D[nt][i] = run[nt][i] * sc;
      }
    }
    if (last) {
      // reduce: O += P F^T over this chunk (4 k-steps of 16 restored channels)
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
          uint32_t f0, f1, f2, f3;
          ldsm_x4(fbase + (uint32_t)((nb * 8 * fs + c0 + kp * 32) * 2), f0, f1, f2, f3);
          mma16816(O[nb], pa[0][0], pa[0][1], pa[0][2], pa[0][3], f0, f1);
          mma16816(O[nb], pa[1][0], pa[1][1], pa[1][2], pa[1][3], f2, f3);
        }
      }
      if (cur.ch == nch - 1) {
        const int64_t m0 = cur.blk * 16 + g, m1 = m0 + 8;
#pragma unroll
        for (int nb = 0; nb < NO; ++nb) {
          const int col = nb * 8 + 2 * t4;
          if (m0 < d.npix) *reinterpret_cast<uint32_t*>(y + m0 * d.Nout + col) = pk2(O[nb][0], O[nb][1]);
          if (m1 < d.npix) *reinterpret_cast<uint32_t*>(y + m1 * d.Nout + col) = pk2(O[nb][2], O[nb][3]);
        }
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

// 64-channel, rank <= 16 groups (VGG's block-1/2 groups, ResNet's stage-1 in-block
// groups, the stem-restore copies): every operand but A is register-resident
// for the whole kernel -- restore weights (16 regs), fconv weights, biases --
// and the bias enters through the MMA's C operand (D = A B + bias), so a
// 16-pixel block costs ~12 MMAs + ReLU / re-pack, about a third of the
// instructions of the generic lean path.

__device__ __forceinline__ void mma16816c(float (&dd)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                          uint32_t b0, uint32_t b1, float c0, float c1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0, %1, %2, %3}, {%4, %5, %6, %7}, {%8, %9}, "
      "{%10, %11, %10, %11};"
      : "=f"(dd[0]), "=f"(dd[1]), "=f"(dd[2]), "=f"(dd[3])
      : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1), "f"(c0), "f"(c1));
}

template <int NO, bool POOL, int kL64Warps = POOL ? 8 : 16>   // pooled: run[] needs > 128 registers
__global__ void __launch_bounds__(32 * kL64Warps, 1) mma_lean64_kernel(const __grid_constant__ MmaChainDesc d,
                                                                       RunPtrs p, const uint16_t* __restrict__ tcw) {
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
  const float* fb = reinterpret_cast<const float*>(smem + (size_t)d.blob_bf16 * 2) + d.bias[0];
  const MmaTerm& T = d.term[0];
  const uint32_t* r = reinterpret_cast<const uint32_t*>(p.arena + T.r.off);
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.arena + d.y.off);
  const int rs = T.Rp + 8, fs = d.Cpad + 8;
  const int lq = lane >> 3, lr = lane & 7;
  // register-resident operands: restore B fragments, fconv B fragments, biases
  uint32_t wb[8][2], fw[NO][4][2];
  float bias[8][2];
#pragma unroll
  for (int np = 0; np < 4; ++np)
    ldsm_x4(s_u32(blob + T.w + (np * 16 + (lq >> 1) * 8 + lr) * rs + (lq & 1) * 8), wb[2 * np][0], wb[2 * np][1],
            wb[2 * np + 1][0], wb[2 * np + 1][1]);
#pragma unroll
  for (int nb = 0; nb < NO; ++nb)
#pragma unroll
    for (int kp = 0; kp < 2; ++kp)
      ldsm_x4(s_u32(blob + d.f + (nb * 8 + lr) * fs + kp * 32 + lq * 8), fw[nb][2 * kp][0], fw[nb][2 * kp][1],
              fw[nb][2 * kp + 1][0], fw[nb][2 * kp + 1][1]);
#pragma unroll
  for (int nt = 0; nt < 8; ++nt) {
    const float2 b = *reinterpret_cast<const float2*>(fb + nt * 8 + 2 * t4);
    bias[nt][0] = b.x;
    bias[nt][1] = b.y;
  }
  const int relu = d.relu[0];
  const int taps = POOL ? d.taps : 1;
  const int64_t nw = (int64_t)gridDim.x * kL64Warps;
  auto advance = [&](LeanCursor& u) {
    if (++u.tap == taps) {
      u.tap = 0;
      u.blk += nw;
      if (u.blk < d.nblocks) lean_set_block(d, u, g);
    }
  };
  LeanCursor cur{};
  cur.blk = (int64_t)blockIdx.x * kL64Warps + warp;
  if (cur.blk < d.nblocks) lean_set_block(d, cur, g);
  LeanCursor pf = cur;
  uint32_t a[1][4], an[1][4], ann[1][4];
  if (pf.blk < d.nblocks) lean_load_a<1>(a, d, r, pf, T.R, g, t4);
  advance(pf);
  if (pf.blk < d.nblocks) lean_load_a<1>(an, d, r, pf, T.R, g, t4);
  advance(pf);
  float run[POOL ? 8 : 1][4];
  const float sc = d.pool == 2 ? 1.f / (float)d.taps : 1.f;
  for (; cur.blk < d.nblocks; advance(cur)) {
    if (pf.blk < d.nblocks) lean_load_a<1>(ann, d, r, pf, T.R, g, t4);
    advance(pf);
    float D[8][4];
#pragma unroll
    for (int nt = 0; nt < 8; ++nt)
      mma16816c(D[nt], a[0][0], a[0][1], a[0][2], a[0][3], wb[nt][0], wb[nt][1], bias[nt][0], bias[nt][1]);
    if (relu) {
#pragma unroll
      for (int nt = 0; nt < 8; ++nt)
#pragma unroll
        for (int i = 0; i < 4; ++i) D[nt][i] = act_apply(D[nt][i], relu);
    }
    bool last = true;
    if constexpr (POOL) {
      float n0 = 0.f, n1 = 0.f;
      if (d.pool == 1) {
        n0 = lean_tap_valid(d, cur, 0) ? 0.f : -INFINITY;
        n1 = lean_tap_valid(d, cur, 1) ? 0.f : -INFINITY;
      }
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) {
        const float x[4] = {D[nt][0] + n0, D[nt][1] + n0, D[nt][2] + n1, D[nt][3] + n1};
#pragma unroll
        for (int i = 0; i < 4; ++i)
          run[nt][i] = cur.tap == 0 ? x[i] : d.pool == 1 ? fmaxf(run[nt][i], x[i]) : run[nt][i] + x[i];
      }
      last = cur.tap == taps - 1;
      if (last) {
#pragma unroll
        for (int nt = 0; nt < 8; ++nt)
#pragma unroll
          for (int i = 0; i < 4; ++i) D[nt][i] = run[nt][i] * sc;
      }
    }
    if (last) {
      float O[NO][4];
#pragma unroll
      for (int ks = 0; ks < 4; ++ks) {
        const uint32_t p0 = pk2(D[2 * ks][0], D[2 * ks][1]), p1 = pk2(D[2 * ks][2], D[2 * ks][3]);
        const uint32_t p2 = pk2(D[2 * ks + 1][0], D[2 * ks + 1][1]), p3 = pk2(D[2 * ks + 1][2], D[2 * ks + 1][3]);
#pragma unroll
        for (int nb = 0; nb < NO; ++nb) {
          if (ks == 0)
            mma16816c(O[nb], p0, p1, p2, p3, fw[nb][0][0], fw[nb][0][1], 0.f, 0.f);
          else
            mma16816(O[nb], p0, p1, p2, p3, fw[nb][ks][0], fw[nb][ks][1]);
        }
      }
      const int64_t m0 = cur.blk * 16 + g, m1 = m0 + 8;
#pragma unroll
      for (int nb = 0; nb < NO; ++nb) {
        const int col = nb * 8 + 2 * t4;
        if (m0 < d.npix) *reinterpret_cast<uint32_t*>(y + m0 * d.Nout + col) = pk2(O[nb][0], O[nb][1]);
        if (m1 < d.npix) *reinterpret_cast<uint32_t*>(y + m1 * d.Nout + col) = pk2(O[nb][2], O[nb][3]);
      }
    }
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      a[0][i] = an[0][i];
      an[0][i] = ann[0][i];
    }
  }
}

template <int NO, bool POOL>
void launch_lean64_t(const MmaChainDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  static bool configured = false;
  static int sms = 148;
  if (!configured) {
    cudaFuncSetAttribute(mma_lean64_kernel<NO, POOL>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    configured = true;
  }
  constexpr int kW = POOL ? 8 : 16;
  const int grid = (int)std::min<int64_t>((d.nblocks + kW - 1) / kW, (int64_t)sms);
  launch_pdl(mma_lean64_kernel<NO, POOL>, dim3(grid), dim3(32 * kW), d.blob_bytes, s, d, p, tcw);
}

template <int KS, int NO>
void launch_lean_t(const MmaChainDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  static bool configured = false;
  static int sms = 148;
  if (!configured) {
    cudaFuncSetAttribute(mma_lean_kernel<KS, NO>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    configured = true;
  }
  const int grid = (int)std::min<int64_t>((d.nblocks + kLeanWarps - 1) / kLeanWarps, (int64_t)sms);
  launch_pdl(mma_lean_kernel<KS, NO>, dim3(grid), dim3(32 * kLeanWarps), d.blob_bytes, s, d, p, tcw);
}

}  // namespace

bool mma_lean_ok(const MmaChainDesc& d) {
  return (d.pool != 2 || d.pp == 0) && d.n_levels == 1 && d.n_terms == 1 && d.term[0].c0 == 0 && d.term[0].C == d.C &&
         d.C % 64 == 0 && d.Cpad == d.C && d.term[0].Rp <= 32 && d.Nout <= 32 && d.blob_bytes <= 200 * 1024;
}

void launch_mma_chain(const MmaChainDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  // register-resident 64-channel variant; pooled groups stay on the generic lean path
  // (their running max needs > 128 registers: 8 warps per SM measured slower)
  if (mma_lean_ok(d) && d.Cpad == 64 && d.term[0].Rp == 16 && d.Nout <= 16 && !d.pool) {
    if (d.Nout <= 8) return launch_lean64_t<1, false>(d, tcw, p, s);
    return launch_lean64_t<2, false>(d, tcw, p, s);
  }
  if (mma_lean_ok(d)) {
    const int ks = d.term[0].Rp / 16, no = (d.Nout + 7) / 8;
#define TEMCO_LEAN_CASE(k, n) \
    if (ks == k && no == n) return launch_lean_t<k, n>(d, tcw, p, s);
    TEMCO_LEAN_CASE(1, 1) TEMCO_LEAN_CASE(1, 2) TEMCO_LEAN_CASE(1, 3) TEMCO_LEAN_CASE(1, 4)
    TEMCO_LEAN_CASE(2, 1) TEMCO_LEAN_CASE(2, 2) TEMCO_LEAN_CASE(2, 3) TEMCO_LEAN_CASE(2, 4)
#undef TEMCO_LEAN_CASE
  }
  const int no = d.Nout <= 32 ? 4 : d.Nout <= 64 ? 8 : 16;
  if (d.pool) {
    if (no == 4) launch_t<64, 4, true>(d, tcw, p, s);
    else if (no == 8) launch_t<64, 8, true>(d, tcw, p, s);
    else launch_t<64, 16, true>(d, tcw, p, s);
    return;
  }
  if (d.CH == 64) {
    if (no == 4) launch_t<64, 4, false>(d, tcw, p, s);
    else if (no == 8) launch_t<64, 8, false>(d, tcw, p, s);
    else launch_t<64, 16, false>(d, tcw, p, s);
  } else {
    if (no == 4) launch_t<128, 4, false>(d, tcw, p, s);
    else if (no == 8) launch_t<128, 8, false>(d, tcw, p, s);
    else launch_t<128, 16, false>(d, tcw, p, s);
  }
}

}  // namespace temco
