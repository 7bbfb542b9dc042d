// tcgen05 fused restore-chain -> BN -> add -> ReLU -> reduce kernel (sm_100a).
//
// One fused group computes, per 128-pixel tile,
//     t_l = act_l( sum_{j in l} r_j Lhat_j^T + b_l + t_{l-1} ),  out = t_D F^T
// with the C-wide t never leaving the SM:
//   GEMM1  TMA (r_j atom [128 x 64], Lhat_j atom [Cc x 64]) -> SMEM ring ->
//          tcgen05.mma (M=128, N=Cc, K=16) -> TMEM accumulator (Cc fp32 columns)
//   level epilogue: TMEM -> registers, + b_l, ReLU, -> TMEM (tcgen05.st) so the
//          next level's MMAs accumulate on top of t_{l-1}; after the last level
//          the bf16 tile P = t_D is written to SMEM in the SW128 K-major layout
//   GEMM2  tcgen05.mma (A = P from SMEM, B = F atom via TMA) -> TMEM (Np columns),
//          accumulated over the C chunks
//   output epilogue: TMEM -> registers -> bf16 -> global.
// Warp roles (192 threads, persistent over tiles): warps 0-3 epilogue (warp w
// owns TMEM lanes 32w..32w+31 = pixel rows), warp 4 TMA producer, warp 5 MMA
// issuer.  Two TMEM accumulators (chunks c, c+1) let the MMA of one chunk
// overlap the epilogue of the other.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cmath>
#include <set>

#include "chain_parse.h"
#include "tc.h"
#include "tc_ptx.cuh"

namespace temco {

// ===========================================================================
// host: lowering of a fused group into a level chain
// ===========================================================================
namespace {
using namespace chainp;

uint16_t to_bf16(float f) {
  uint32_t u;
  memcpy(&u, &f, 4);
  u += 0x7FFF + ((u >> 16) & 1);
  return (uint16_t)(u >> 16);
}

int64_t push_bf16(std::vector<uint16_t>& pool, const std::vector<float>& v) {
  while (pool.size() % 512) pool.push_back(0);   // 1024-byte aligned blocks (TMA base alignment)
  int64_t off = (int64_t)pool.size();
  for (float f : v) pool.push_back(to_bf16(f));
  return off;
}

int64_t push_f32(std::vector<float>& pool, const std::vector<double>& v) {
  while (pool.size() % 4) pool.push_back(0.f);
  int64_t off = (int64_t)pool.size();
  for (double x : v) pool.push_back((float)x);
  while (pool.size() % 4) pool.push_back(0.f);
  return off;
}

}  // namespace

bool tc_lower_chain(const IR& ir, const Step& s, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                    std::vector<float>& params, TcChainDesc& d) {
  const Node& root = ir.nodes[s.out];
  const bool gap = root.op == OP_GAP;
  if (root.role != ROLE_FCONV && !gap) return false;
  const int tsrc = ir.oin[s.out][0];
  const Node& tn = ir.nodes[tsrc];
  const int C = tn.C, Nout = gap ? 16 : root.C;
  if (Nout % 8 || Nout > 256) return false;
  if (gap && tn.H * tn.W > 128) return false;
  // pooled chain (Listing 1 with p >= 2): root fconv <- max/avg pool <- level chain
  int pool = 0, pk = 1, ps = 1, pp = 0, csrc = tsrc;
  if (!gap && (tn.op == OP_MAXPOOL || tn.op == OP_AVGPOOL) && s.members.size() > 2) {
    pool = tn.op == OP_MAXPOOL ? 1 : 2;
    pk = tn.kh; ps = tn.sh; pp = tn.ph;
    csrc = ir.oin[tsrc][0];
  }
  const Node& cn = ir.nodes[csrc];
  ChainParser P{ir, std::set<int>(s.members.begin(), s.members.end()), C, {}, cn.H, cn.W};
  P.members.erase(s.out);
  if (pool) P.members.erase(tsrc);
  std::vector<PLevel> levels;
  if (!P.chain(csrc, levels)) return false;
  if (P.visited != P.members) return false;          // every member must be part of the chain form
  int nterms = 0;
  for (auto& L : levels) nterms += (int)L.terms.size();
  if ((int)levels.size() > kTcMaxLevels || nterms > kTcMaxTerms) return false;
  // term inputs: bf16 reduced tensors in the arena, ranks % 8 == 0
  for (auto& L : levels)
    for (auto& t : L.terms) {
      const int r = ir.oin[t.lconv][0];
      const Loc& l = loc.at(r);
      if (l.where != W_ARENA || l.dtype != DT_BF16 || ir.nodes[r].C % 8) return false;
    }
  const Loc& yl = loc.at(s.out);
  if (yl.where != W_ARENA || yl.dtype != DT_BF16) return false;

  d = TcChainDesc();
  d.C = C;
  d.Cc = (C <= 64 || pool) ? 64 : 128;
  d.gather = pool ? 1 : 0;
  d.pool = pool; d.pk = pk; d.ps = ps; d.pp = pp; d.taps = pk * pk;
  d.Hin = cn.H; d.Win = cn.W; d.Ho = tn.H; d.Wo = tn.W;
  d.Cpad = (C + d.Cc - 1) / d.Cc * d.Cc;
  d.nchunks = d.Cpad / d.Cc;
  d.Nout = Nout;
  d.Np = (Nout + 15) / 16 * 16;
  d.npix = (int64_t)ir.batch * tn.H * tn.W;
  d.nimg = ir.batch;
  d.gap = gap ? 1 : 0;
  d.hw = tn.H * tn.W;
  if (gap) {
    d.ipt = 128 / d.hw;
    d.rows_per_tile = d.ipt * d.hw;
    d.ntiles = (ir.batch + d.ipt - 1) / d.ipt;
  } else {
    d.ipt = 0;
    d.rows_per_tile = 128;
    d.ntiles = (int)((d.npix + 127) / 128);
  }
  d.y = yl;
  d.n_levels = (int)levels.size();
  int64_t flops_terms = 0, bytes_terms = 0;
  int j = 0;
  for (int l = 0; l < d.n_levels; ++l) {
    const PLevel& L = levels[l];
    d.relu[l] = L.relu ? 1 : 0;
    std::vector<double> bias(d.Cpad, 0.0);
    std::copy(L.bias.begin(), L.bias.end(), bias.begin());
    d.bias[l] = push_f32(params, bias);
    for (const PTerm& t : L.terms) {
      const Node& lc = ir.nodes[t.lconv];
      const int r = ir.oin[t.lconv][0];
      const int R = ir.nodes[r].C;
      TcTerm& T = d.term[j++];
      T.r = loc.at(r);
      T.R = R;
      T.Rp = (R + 63) / 64 * 64;
      T.c0 = t.c0;
      T.C = lc.C;
      std::vector<float> w((size_t)d.Cpad * T.Rp, 0.f);
      for (int c = 0; c < lc.C; ++c)
        for (int k = 0; k < R; ++k)
          w[(size_t)(t.c0 + c) * T.Rp + k] = (float)(t.scale[c] * (*lc.w)[(size_t)c * R + k]);
      T.w = push_bf16(tcw, w);
      flops_terms += 2LL * lc.C * R;
      bytes_terms += 2LL * R;
    }
    d.lvl_end[l] = j;
  }
  d.n_terms = j;
  d.Fb = -1;
  if (gap) {
    d.F = 0;
    d.alg_flops = d.npix * (flops_terms + C);
    d.alg_bytes = d.npix * bytes_terms + 2LL * ir.batch * C;
  } else {
    std::vector<float> f((size_t)d.Np * d.Cpad, 0.f);
    for (int o = 0; o < Nout; ++o)
      for (int c = 0; c < C; ++c) f[(size_t)o * d.Cpad + c] = (*root.w)[(size_t)o * C + c];
    d.F = push_bf16(tcw, f);
    if (root.b) {
      std::vector<double> fb(root.b->begin(), root.b->end());
      d.Fb = push_f32(params, fb);
    }
    const int64_t nin = (int64_t)ir.batch * cn.H * cn.W;   // chain evaluated once per input pixel
    d.alg_flops = nin * flops_terms + d.npix * 2LL * Nout * C;
    d.alg_bytes = nin * bytes_terms + d.npix * 2LL * Nout;
  }
  // shared memory: ring of (A 16 KB | B slot) stages + two P tiles + barriers
  d.slot_b = std::max(d.Cc, d.Np) * 128;
  const int pbytes = 128 * d.Cc * 2;
  const int budget = 227 * 1024 - 1024 /*align*/ - 512 /*barriers*/ - 2 * pbytes;
  d.stages = std::min(6, budget / (16384 + d.slot_b));
  if (d.stages < 2) return false;
  d.smem_bytes = 1024 + d.stages * (16384 + d.slot_b) + 2 * pbytes + 512;
  const int cols = 2 * d.Cc + d.Np;
  d.tmem_cols = cols <= 32 ? 32 : cols <= 64 ? 64 : cols <= 128 ? 128 : cols <= 256 ? 256 : 512;
  return true;
}

bool tc_finalize(size_t n, const std::function<TcChainDesc*(size_t)>& get, char* arena, uint16_t* tcw,
                 std::string& err) {
  static PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
  bool any = false;
  for (size_t i = 0; i < n; ++i) any |= get(i) != nullptr;
  if (!any) return true;
  if (!encode) {
    cudaDriverEntryPointQueryResult q;
    void* fn = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn) {
      err = "cuTensorMapEncodeTiled unavailable";
      return false;
    }
    encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  }
  auto make = [&](unsigned char* dst, void* base, uint64_t inner, uint64_t outer, uint32_t box_outer) {
    cuuint64_t dims[2] = {inner, outer};
    cuuint64_t strides[1] = {inner * 2};
    cuuint32_t box[2] = {64, box_outer};
    cuuint32_t es[2] = {1, 1};
    CUresult r = encode(reinterpret_cast<CUtensorMap*>(dst), CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, base, dims, strides,
                        box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
  };
  for (size_t i = 0; i < n; ++i) {
    TcChainDesc* d = get(i);
    if (!d) continue;
    for (int j = 0; j < d->n_terms; ++j) {
      TcTerm& t = d->term[j];
      if (!make(t.tmap, arena + t.r.off, (uint64_t)t.R, (uint64_t)d->npix, 128) ||
          !make(t.wmap, tcw + t.w, (uint64_t)t.Rp, (uint64_t)d->Cpad, (uint32_t)d->Cc)) {
        err = "cuTensorMapEncodeTiled failed (term)";
        return false;
      }
    }
    if (!d->gap && !make(d->fmap, tcw + d->F, (uint64_t)d->Cpad, (uint64_t)d->Np, (uint32_t)d->Np)) {
      err = "cuTensorMapEncodeTiled failed (F)";
      return false;
    }
  }
  return true;
}

// ===========================================================================
// device
// ===========================================================================
namespace {
using namespace ptx;

__device__ __forceinline__ bool term_hits(const TcTerm& t, int c, int Cc) {
  return t.c0 < (c + 1) * Cc && t.c0 + t.C > c * Cc;
}

constexpr int kThreads = 320;   // warps 0-3 epilogue, 4 TMA producer, 5 MMA, 6-9 gather (gather mode)
constexpr int kSlotA = 16384;

// The MMA work of one tile is a sequence of "units": chunk c of the restored
// width (and, for a pooled chain, tap tau of the pooling window).  Units are
// processed in pairs (two TMEM accumulators) -- consecutive chunks, or
// consecutive taps of one chunk -- and every role walks the same order:
//   for pair: for level l: for unit in pair: G1(unit, l) [+ epilogue E(unit, l)]
//             then G2 for every chunk whose restored values are final.
struct PairIter {
  int c0, t0, nb;
};

__device__ __forceinline__ void unit_of(const TcChainDesc& d, const PairIter& it, int bi, int& c, int& tap) {
  if (d.pool) {
    c = it.c0;
    tap = it.t0 + bi;
  } else {
    c = it.c0 + bi;
    tap = 0;
  }
}

#define FOR_PAIRS(d, it)                                                                            \
  for (PairIter it{0, 0, 0}; it.c0 < (d).nchunks;                                                   \
       (d).pool ? ((it.t0 += 2) >= (d).taps ? (it.t0 = 0, ++it.c0) : 0) : (it.c0 += 2))             \
    if ((it.nb = (d).pool ? min(2, (d).taps - it.t0) : min(2, (d).nchunks - it.c0)), true)

// chunks whose G2 follows this pair: non-pool -> c0 .. c0+nb-1; pool -> c0 after its last tap
__device__ __forceinline__ int g2_count(const TcChainDesc& d, const PairIter& it) {
  if (d.gap) return 0;
  if (d.pool) return it.t0 + it.nb == d.taps ? 1 : 0;
  return it.nb;
}

__global__ void __launch_bounds__(kThreads, 1) tc_chain_kernel(const __grid_constant__ TcChainDesc d, RunPtrs p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  const int S = d.stages;
  const int slot = kSlotA + d.slot_b;
  const int Cc = d.Cc;
  const int pbytes = 128 * Cc * 2;
  uint8_t* ring = smem;
  uint8_t* pbuf = ring + S * slot;
  uint64_t* bars = reinterpret_cast<uint64_t*>(pbuf + 2 * pbytes);
  uint64_t* full = bars;
  uint64_t* empty = bars + S;
  uint64_t* acc_full = bars + 2 * S;
  uint64_t* acc_empty = acc_full + 2;
  uint64_t* p_full = acc_empty + 2;
  uint64_t* p_empty = p_full + 2;
  uint64_t* out_full = p_empty + 2;
  uint64_t* out_empty = out_full + 1;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(out_empty + 1);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], d.gather ? 33 : 1);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&acc_full[b], 1);
      mbar_init(&acc_empty[b], 128);
      mbar_init(&p_full[b], 128);
      mbar_init(&p_empty[b], 1);
    }
    mbar_init(out_full, 1);
    mbar_init(out_empty, 128);
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

  if (warp == 4) {
    // ------------------------------------------------------------ TMA producer
    if (lane == 0) {
      int stage = 0;
      uint32_t phase = 0;
      const uint32_t bytes_b = Cc * 128, bytes_a = d.gather ? 0 : kSlotA, bytes_f = d.Np * 128;
      for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x) {
        const int m0 = tile * d.rows_per_tile;
        FOR_PAIRS(d, it) {
          for (int l = 0; l < d.n_levels; ++l)
            for (int bi = 0; bi < it.nb; ++bi) {
              int c, tap;
              unit_of(d, it, bi, c, tap);
              for (int j = l ? d.lvl_end[l - 1] : 0; j < d.lvl_end[l]; ++j) {
                const TcTerm& t = d.term[j];
                if (!term_hits(t, c, Cc)) continue;
                for (int ka = 0; ka < t.Rp / 64; ++ka) {
                  mbar_wait(&empty[stage], phase ^ 1);
                  mbar_expect_tx(&full[stage], bytes_a + bytes_b);
                  uint8_t* sa = ring + stage * slot;
                  if (!d.gather) tma_load_2d(sa, t.tmap, &full[stage], ka * 64, m0);
                  tma_load_2d(sa + kSlotA, t.wmap, &full[stage], ka * 64, c * Cc);
                  if (++stage == S) stage = 0, phase ^= 1;
                }
              }
            }
          for (int q = 0; q < g2_count(d, it); ++q) {
            const int c = it.c0 + (d.pool ? 0 : q);
            for (int a = 0; a < Cc / 64; ++a) {
              mbar_wait(&empty[stage], phase ^ 1);
              mbar_expect_tx(&full[stage], bytes_f);
              tma_load_2d(ring + stage * slot + kSlotA, d.fmap, &full[stage], c * Cc + a * 64, 0);
              if (++stage == S) stage = 0, phase ^= 1;
            }
          }
        }
      }
    }
  } else if (warp >= 6) {
    // ------------------------------------------------------------ gather producer (A rows)
    // warp-per-stage: gather warp gw fills every 4th stage of the ring (lane
    // owns rows lane + 32 i), so 4 stages of cp.async are in flight at once
    if (d.gather) {
      const int gw = warp - 6;
      int64_t kseq = 0;
      auto next = [&](int& stage, uint32_t& phase) {
        stage = (int)(kseq % S);
        phase = (uint32_t)((kseq / S) & 1);
        return (int)((kseq++) & 3) == gw;
      };
      for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x) {
        int ho[4], wo[4], nn[4];
        bool mv[4];
        const int hw = d.Ho * d.Wo;
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int64_t m = (int64_t)tile * d.rows_per_tile + lane + 32 * i;
          mv[i] = m < d.npix;
          nn[i] = mv[i] ? (int)(m / hw) : 0;
          const int rem = mv[i] ? (int)(m % hw) : 0;
          ho[i] = rem / d.Wo;
          wo[i] = rem % d.Wo;
        }
        FOR_PAIRS(d, it) {
          for (int l = 0; l < d.n_levels; ++l)
            for (int bi = 0; bi < it.nb; ++bi) {
              int c, tap;
              unit_of(d, it, bi, c, tap);
              for (int j = l ? d.lvl_end[l - 1] : 0; j < d.lvl_end[l]; ++j) {
                const TcTerm& t = d.term[j];
                if (!term_hits(t, c, Cc)) continue;
                const uint8_t* rbase = reinterpret_cast<const uint8_t*>(p.arena + t.r.off);
                for (int ka = 0; ka < t.Rp / 64; ++ka) {
                  int stage;
                  uint32_t phase;
                  if (!next(stage, phase)) continue;
                  mbar_wait(&empty[stage], phase ^ 1);
#pragma unroll
                  for (int i = 0; i < 4; ++i) {
                    const int row = lane + 32 * i;
                    const int hi = ho[i] * d.ps - d.pp + tap / d.pk, wi = wo[i] * d.ps - d.pp + tap % d.pk;
                    const bool valid = mv[i] && hi >= 0 && hi < d.Hin && wi >= 0 && wi < d.Win;
                    const int64_t pix = ((int64_t)nn[i] * d.Hin + hi) * d.Win + wi;
                    uint8_t* dst = ring + stage * slot + row * 128;
#pragma unroll
                    for (int q = 0; q < 8; ++q) {
                      const int k0 = ka * 64 + q * 8;
                      const bool ok = valid && k0 < t.R;
                      cp_async16(dst + ((q ^ (row & 7)) * 16), ok ? rbase + (pix * t.R + k0) * 2 : rbase, ok ? 16u : 0u);
                    }
                  }
                  cp_async_arrive(&full[stage]);
                }
              }
            }
          for (int q = 0; q < g2_count(d, it) * (Cc / 64); ++q) {
            int stage;
            uint32_t phase;
            if (!next(stage, phase)) continue;
            mbar_wait(&empty[stage], phase ^ 1);
            cp_async_arrive(&full[stage]);
          }
        }
      }
    }
  } else if (warp == 5) {
    // ------------------------------------------------------------ MMA issuer
    if (lane == 0) {
      int stage = 0;
      uint32_t phase = 0;
      uint32_t acc_use[2] = {0, 0}, p_use[2] = {0, 0}, tile_iter = 0;
      const uint32_t id1 = idesc_bf16(128, Cc), id2 = idesc_bf16(128, d.Np);
      const uint32_t tout = tbase + 2 * Cc;
      for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x) {
        FOR_PAIRS(d, it) {
          for (int l = 0; l < d.n_levels; ++l)
            for (int bi = 0; bi < it.nb; ++bi) {
              int c, tap;
              unit_of(d, it, bi, c, tap);
              mbar_wait(&acc_empty[bi], (acc_use[bi] & 1) ^ 1);
              tc_fence_after();
              const uint32_t tacc = tbase + bi * Cc;
              bool first = (l == 0);
              for (int j = l ? d.lvl_end[l - 1] : 0; j < d.lvl_end[l]; ++j) {
                const TcTerm& t = d.term[j];
                if (!term_hits(t, c, Cc)) continue;
                for (int ka = 0; ka < t.Rp / 64; ++ka) {
                  mbar_wait(&full[stage], phase);
                  if (d.gather) fence_proxy_async();
                  tc_fence_after();
                  const uint32_t sa = smem_u32(ring + stage * slot);
                  const int nk = min(4, (t.R - ka * 64 + 15) / 16);
                  for (int k = 0; k < nk; ++k) {
                    mma_bf16(tacc, umma_desc(sa + 32 * k), umma_desc(sa + kSlotA + 32 * k), id1, first ? 0u : 1u);
                    first = false;
                  }
                  mma_commit(&empty[stage]);
                  if (++stage == S) stage = 0, phase ^= 1;
                }
              }
              mma_commit(&acc_full[bi]);
              ++acc_use[bi];
            }
          for (int q = 0; q < g2_count(d, it); ++q) {
            const int c = it.c0 + (d.pool ? 0 : q);
            const int pb = c & 1;
            mbar_wait(&p_full[pb], p_use[pb] & 1);
            tc_fence_after();
            if (c == 0) {
              mbar_wait(out_empty, (tile_iter & 1) ^ 1);
              tc_fence_after();
            }
            const uint32_t pa = smem_u32(pbuf + pb * pbytes);
            for (int a = 0; a < Cc / 64; ++a) {
              mbar_wait(&full[stage], phase);
              tc_fence_after();
              const uint32_t sb = smem_u32(ring + stage * slot + kSlotA);
              for (int k = 0; k < 4; ++k)
                mma_bf16(tout, umma_desc(pa + a * 16384 + 32 * k), umma_desc(sb + 32 * k), id2,
                         (c > 0 || a > 0 || k > 0) ? 1u : 0u);
              mma_commit(&empty[stage]);
              if (++stage == S) stage = 0, phase ^= 1;
            }
            mma_commit(&p_empty[pb]);
            ++p_use[pb];
          }
        }
        if (!d.gap) mma_commit(out_full);
        ++tile_iter;
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue (128 threads)
    const int row = threadIdx.x;                       // pixel row in the tile == TMEM lane
    const uint32_t lane_off = (uint32_t)(warp * 32) << 16;
    uint32_t acc_use[2] = {0, 0}, p_use[2] = {0, 0}, tile_iter = 0;
    __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.arena + d.y.off);
    float run[64];                                     // pooled values of the current chunk (pool mode, Cc = 64)
    for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x) {
      const int64_t m = (int64_t)tile * d.rows_per_tile + row;
      int ho = 0, wo = 0;
      if (d.pool) {
        const int rem = (int)(m % (d.Ho * d.Wo));
        ho = rem / d.Wo;
        wo = rem % d.Wo;
      }
      FOR_PAIRS(d, it) {
        for (int l = 0; l < d.n_levels; ++l) {
          const bool last = l == d.n_levels - 1;
          const bool relu = d.relu[l] != 0;
          for (int bi = 0; bi < it.nb; ++bi) {
            int c, tap;
            unit_of(d, it, bi, c, tap);
            mbar_wait(&acc_full[bi], acc_use[bi] & 1);
            ++acc_use[bi];
            tc_fence_after();
            const int pb = c & 1;
            const bool writes_p = last && !d.gap && (!d.pool || tap == d.taps - 1);
            if (writes_p) {
              mbar_wait(&p_empty[pb], (p_use[pb] & 1) ^ 1);
              ++p_use[pb];
            }
            const float* bias = p.params + d.bias[l] + (int64_t)c * Cc;
            uint8_t* P = pbuf + pb * pbytes;
            if (d.pool && last) {
              // pooled chain: fold this tap into the running max / sum (Cc == 64)
              const int hi = ho * d.ps - d.pp + tap / d.pk, wi = wo * d.ps - d.pp + tap % d.pk;
              const bool valid = hi >= 0 && hi < d.Hin && wi >= 0 && wi < d.Win;
#pragma unroll
              for (int g = 0; g < 2; ++g) {
                uint32_t v[32];
                tmem_ld32(tbase + lane_off + bi * Cc + g * 32, v);
                tmem_wait_ld();
#pragma unroll
                for (int i = 0; i < 32; ++i) {
                  float x = __uint_as_float(v[i]) + __ldg(bias + g * 32 + i);
                  x = relu ? fmaxf(x, 0.f) : x;
                  float& r = run[g * 32 + i];
                  if (d.pool == 1)
                    r = tap == 0 ? (valid ? x : -INFINITY) : (valid ? fmaxf(r, x) : r);
                  else
                    r = tap == 0 ? x : r + x;
                }
              }
              if (writes_p) {
                const float scale = d.pool == 2 ? 1.f / (float)d.taps : 1.f;
#pragma unroll
                for (int q = 0; q < 8; ++q) {
                  uint4 pk;
                  pk.x = pack_bf16(run[8 * q + 0] * scale, run[8 * q + 1] * scale);
                  pk.y = pack_bf16(run[8 * q + 2] * scale, run[8 * q + 3] * scale);
                  pk.z = pack_bf16(run[8 * q + 4] * scale, run[8 * q + 5] * scale);
                  pk.w = pack_bf16(run[8 * q + 6] * scale, run[8 * q + 7] * scale);
                  *reinterpret_cast<uint4*>(P + row * 128 + ((q ^ (row & 7)) * 16)) = pk;
                }
              }
            } else {
              for (int g = 0; g < Cc / 32; ++g) {
                const uint32_t ta = tbase + lane_off + bi * Cc + g * 32;
                uint32_t v[32];
                tmem_ld32(ta, v);
                tmem_wait_ld();
                float f[32];
#pragma unroll
                for (int i = 0; i < 32; ++i) {
                  float x = __uint_as_float(v[i]) + __ldg(bias + g * 32 + i);
                  f[i] = relu ? fmaxf(x, 0.f) : x;
                }
                if (!last) {
#pragma unroll
                  for (int i = 0; i < 32; ++i) v[i] = __float_as_uint(f[i]);
                  tmem_st32(ta, v);
                } else if (d.gap) {
                  // GAP root: per-image column means of this 32-column group; tiles
                  // hold whole images so the reduction order is fixed (deterministic)
                  float* red = reinterpret_cast<float*>(pbuf);
#pragma unroll
                  for (int i = 0; i < 32; ++i) red[row * 32 + ((i + row) & 31)] = f[i];
                  asm volatile("bar.sync 1, 128;" ::: "memory");
                  for (int idx = row; idx < d.ipt * 32; idx += 128) {
                    const int ii = idx / 32, col = idx % 32;
                    const int n = tile * d.ipt + ii;
                    float acc = 0.f;
                    for (int r = ii * d.hw; r < (ii + 1) * d.hw; ++r) acc += red[r * 32 + ((col + r) & 31)];
                    const int cg = c * Cc + g * 32 + col;
                    if (n < d.nimg && cg < d.C) y[(int64_t)n * d.C + cg] = __float2bfloat16_rn(acc / (float)d.hw);
                  }
                  asm volatile("bar.sync 1, 128;" ::: "memory");
                } else {
                  const int col = g * 32;                     // within the chunk
                  uint8_t* atom = P + (col / 64) * 16384 + row * 128;
                  const int ch0 = (col % 64) / 8;
#pragma unroll
                  for (int q = 0; q < 4; ++q) {
                    uint4 pk;
                    pk.x = pack_bf16(f[8 * q + 0], f[8 * q + 1]);
                    pk.y = pack_bf16(f[8 * q + 2], f[8 * q + 3]);
                    pk.z = pack_bf16(f[8 * q + 4], f[8 * q + 5]);
                    pk.w = pack_bf16(f[8 * q + 6], f[8 * q + 7]);
                    *reinterpret_cast<uint4*>(atom + (((ch0 + q) ^ (row & 7)) * 16)) = pk;
                  }
                }
              }
              if (!last) tmem_wait_st();
            }
            tc_fence_before();
            mbar_arrive(&acc_empty[bi]);
            if (writes_p) {
              fence_proxy_async();
              mbar_arrive(&p_full[pb]);
            }
          }
        }
      }
      if (d.gap) continue;
      // output epilogue
      mbar_wait(out_full, tile_iter & 1);
      ++tile_iter;
      tc_fence_after();
      for (int g = 0; g < d.Np / 8; ++g) {
        uint32_t v[8];
        tmem_ld8(tbase + lane_off + 2 * Cc + g * 8, v);
        tmem_wait_ld();
        if (m < d.npix && g * 8 < d.Nout) {
          float f[8];
#pragma unroll
          for (int i = 0; i < 8; ++i) f[i] = __uint_as_float(v[i]) + (d.Fb >= 0 ? __ldg(p.params + d.Fb + g * 8 + i) : 0.f);
          uint4 pk;
          pk.x = pack_bf16(f[0], f[1]);
          pk.y = pack_bf16(f[2], f[3]);
          pk.z = pack_bf16(f[4], f[5]);
          pk.w = pack_bf16(f[6], f[7]);
          *reinterpret_cast<uint4*>(y + m * d.Nout + g * 8) = pk;
        }
      }
      tc_fence_before();
      mbar_arrive(out_empty);
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

void launch_tc_chain(const TcChainDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  (void)tcw;
  static bool configured = false;
  static int sms = 0;
  if (!configured) {
    cudaFuncSetAttribute(tc_chain_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    configured = true;
  }
  const int grid = std::min(d.ntiles, sms > 0 ? sms : 148);
  // >= 114 KB of shared memory keeps one CTA per SM (each may own all 512 TMEM columns)
  tc_chain_kernel<<<grid, kThreads, std::max(d.smem_bytes, 116 * 1024), s>>>(d, p);
}

}  // namespace temco
