// tcgen05 CTA-pair fused restore-chain kernel (sm_100a): see pair.h.
//
// Work order (every role walks it): for each 256-pixel pair tile (rows tile*256 +
// cta*128 + [0, 128) on each CTA of a 2-CTA cluster), for each 128-channel unit u
// of the restored width, for each level l:
//   TMA   r_j atom [128 px x aw]  (each CTA its own pixels)             -> ring A
//         Lhat_j atom [64 rows x aw] (each CTA its half of the unit)    -> ring B
//   MMA   cta_group::2, M = 256, N = 128, fresh accumulator a_l in TMEM buffer
//         (global level count mod nbuf): a_l = sum_{j in l} r_j Lhat_j[u]^T
//   epilogue (16 warps per CTA: TMEM lane quarter x 32 columns each), t in registers:
//         t = act_l(a_l + b_l [+ t])   -- the residual add of Fig. 8 / P:L333
//         the buffer is released right after tcgen05.ld, before the math
//   after the last level: P = bf16(t) -> shared memory (SW128 K-major), and one
//   level later (so the tensor pipe never waits for it) the fconv
//         out += P F[:, unit u]^T   (M = 256, N = Np, TMEM columns 128 nbuf ..)
// and after the last unit out -> bf16 -> global.  The C-wide t never reaches
// global memory.
//
// Warp roles (18 warps): 0 TMA producer (both CTAs), 1 TMEM allocator (both) and
// MMA issuer (leader CTA), 2-17 epilogue (both).  Barriers the issuer waits on
// live in the leader CTA (peer arrivals through shared::cluster addresses);
// commits are multicast to both CTAs.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cmath>
#include <cstring>
#include <set>

#include "chain_parse.h"
#include "pair.h"
#include "tc_ptx.cuh"

namespace temco {
namespace pair {

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
  const int64_t off = (int64_t)pool.size();
  for (float f : v) pool.push_back(to_bf16(f));
  return off;
}

constexpr int kSlotA = 16384;            // 128 rows x 64 bf16 (r atom; or an F atom of Np/2 rows)
constexpr int kSlotB = 8192;             // 64 rows x 64 bf16 (this CTA's half of a unit's Lhat atom)
constexpr int kSlot = kSlotA + kSlotB;
constexpr int kPBytes = 128 * kPairWu * 2;   // P: two SW128 atoms of 128 x 64
constexpr int kBarBytes = 1024;

}  // namespace

bool pair_lower_chain(const IR& ir, const Step& s, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                      std::vector<float>& params, PairDesc& d) {
  if (getenv("TEMCO_NO_PAIR")) return false;
  const Node& root = ir.nodes[s.out];
  if (root.role != ROLE_FCONV || root.b) return false;   // fconv factors carry no bias (O1)
  const int tsrc = ir.oin[s.out][0];
  const Node& tn = ir.nodes[tsrc];
  const int C = tn.C, Nout = root.C;
  if (Nout % 8 || (Nout + 15) / 16 * 16 > 256) return false;
  ChainParser P{ir, std::set<int>(s.members.begin(), s.members.end()), C, {}, tn.H, tn.W};
  P.allow_silu = true;
  P.members.erase(s.out);
  std::vector<PLevel> levels;
  if (!P.chain(tsrc, levels)) return false;
  if (P.visited != P.members) return false;
  int nterms = 0;
  for (auto& L : levels) {
    if (!L.pm.empty()) return false;
    for (auto& t : L.terms) {
      if (t.tk != 1 || t.c0 != 0 || ir.nodes[t.lconv].C != C) return false;   // full-width plain terms
      const int r = ir.oin[t.lconv][0];
      const Loc& l = loc.at(r);
      const Node& rn = ir.nodes[r];
      if (l.where != W_ARENA || l.dtype != DT_BF16 || rn.C % 8 || rn.H != tn.H || rn.W != tn.W) return false;
      ++nterms;
    }
  }
  if ((int)levels.size() > kPairMaxLevels || nterms > kPairMaxTerms || nterms == 0) return false;
  const Loc& yl = loc.at(s.out);
  if (yl.where != W_ARENA || yl.dtype != DT_BF16) return false;

  d = PairDesc();
  d.C = C;
  d.Cpad = (C + kPairWu - 1) / kPairWu * kPairWu;
  d.nunits = d.Cpad / kPairWu;
  d.Nout = Nout;
  d.Np = (Nout + 15) / 16 * 16;
  d.nbuf = (512 - d.Np) / kPairWu;   // 3 for Np <= 128, 2 for Np <= 256
  if (d.nbuf < 2) return false;
  d.npix = (int64_t)ir.batch * tn.H * tn.W;
  d.ntiles = (int)((d.npix + 255) / 256);
  d.y = yl;
  d.n_levels = (int)levels.size();
  int64_t flops = 0, bytes = 0;
  while (params.size() % 4) params.push_back(0.f);
  d.lbias = (int64_t)params.size();
  for (int l = 0; l < d.n_levels; ++l) {
    const PLevel& L = levels[l];
    d.act[l] = L.relu ? 1 : L.silu ? 2 : 0;
    d.silu |= L.silu ? 1 : 0;
    for (int c = 0; c < d.Cpad; ++c) params.push_back(c < C ? (float)L.bias[c] : 0.f);
  }
  int j = 0;
  for (int l = 0; l < d.n_levels; ++l) {
    for (const PTerm& t : levels[l].terms) {
      const Node& lc = ir.nodes[t.lconv];
      const int r = ir.oin[t.lconv][0];
      const int R = ir.nodes[r].C;
      PairTerm& T = d.term[j++];
      T.r = loc.at(r);
      T.R = R;
      T.aw = R <= 16 ? 16 : R <= 32 ? 32 : 64;
      T.natoms = (R + T.aw - 1) / T.aw;
      T.Rw = (R + 7) / 8 * 8;
      std::vector<float> w((size_t)d.Cpad * T.Rw, 0.f);
      for (int c = 0; c < C; ++c)
        for (int k = 0; k < R; ++k) w[(size_t)c * T.Rw + k] = (float)(t.scale[c] * (*lc.w)[(size_t)c * R + k]);
      T.w = push_bf16(tcw, w);
      flops += d.npix * 2LL * C * R;
      bytes += d.npix * 2LL * R;
    }
    d.lvl_end[l] = j;
  }
  d.n_terms = j;
  int natoms = 0;
  for (int i = 0; i < j; ++i) natoms += d.term[i].natoms;
  if (natoms > 64) return false;   // the kernel's per-unit atom program holds 64 entries
  std::vector<float> f((size_t)d.Np * d.Cpad, 0.f);
  for (int o = 0; o < Nout; ++o)
    for (int c = 0; c < C; ++c) f[(size_t)o * d.Cpad + c] = (*root.w)[(size_t)o * C + c];
  d.F = push_bf16(tcw, f);
  d.alg_flops = flops + d.npix * 2LL * Nout * C;
  d.alg_bytes = bytes + d.npix * 2LL * Nout;
  // level biases live in shared memory (fp32 [n_levels][Cpad]): L1 is ~empty next to
  // 200+ KB of shared memory, so per-level global bias loads would each cost an L2 trip
  d.bias_bytes = (d.n_levels * d.Cpad * 4 + 1023) / 1024 * 1024;
  const int budget = 227 * 1024 - 1024 /*align*/ - kBarBytes - kPBytes - d.bias_bytes;
  d.stages = std::min(8, budget / kSlot);
  if (d.stages < 3) return false;
  d.smem_bytes = 1024 + d.stages * kSlot + kPBytes + d.bias_bytes + kBarBytes;
  return true;
}

bool pair_finalize(size_t n, const std::function<PairDesc*(size_t)>& get, char* arena, uint16_t* tcw,
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
  auto make = [&](unsigned char* dst, void* base, uint64_t inner, uint64_t outer, uint32_t box_outer, int aw) {
    cuuint64_t dims[2] = {inner, outer};
    cuuint64_t strides[1] = {inner * 2};
    cuuint32_t box[2] = {(cuuint32_t)aw, box_outer};
    cuuint32_t es[2] = {1, 1};
    const CUtensorMapSwizzle sw = aw == 64 ? CU_TENSOR_MAP_SWIZZLE_128B
                                  : aw == 32 ? CU_TENSOR_MAP_SWIZZLE_64B
                                             : CU_TENSOR_MAP_SWIZZLE_32B;
    return encode(reinterpret_cast<CUtensorMap*>(dst), CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, base, dims, strides, box,
                  es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
  };
  for (size_t i = 0; i < n; ++i) {
    PairDesc* d = get(i);
    if (!d) continue;
    for (int j = 0; j < d->n_terms; ++j) {
      PairTerm& t = d->term[j];
      const bool ok = make(t.amap, arena + t.r.off, (uint64_t)t.R, (uint64_t)d->npix, 128, t.aw) &&
                      make(t.wmap, tcw + t.w, (uint64_t)t.Rw, (uint64_t)d->Cpad, 64, t.aw);
      if (!ok) {
        err = "cuTensorMapEncodeTiled failed (pair term)";
        return false;
      }
    }
    if (!make(d->fmap, tcw + d->F, (uint64_t)d->Cpad, (uint64_t)d->Np, (uint32_t)(d->Np / 2), 64)) {
      err = "cuTensorMapEncodeTiled failed (pair F)";
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

#ifdef TEMCO_TRACE
// experiment builds only: cycle accounting of pair 0's MMA issuer and of one epilogue warp
// [launch][0 issuer total, 1 wait full, 2 wait acc_empty, 3 wait p_full, 4 wait out_empty, 5 mma issue,
//          6 commits, 8 epi total, 9 wait acc_full, 10 wait p_empty, 11 tmem ld+arrive, 12 math,
//          13 wait out_full, 14 P write, 15 out store]
__device__ unsigned long long g_pprof[64][16];
__device__ int g_pprof_n;
__device__ int g_pdbg;   // 1: producer issues no TMA (stale operands; timing experiment only)
#define PT0() (_t0 = clock64())
#define PTADD(i) (_acc[i] += clock64() - _t0)
#define PTDECL() long long _t0 = 0, _acc[16] = {0}; const long long _start = clock64()
#define PTSAVE(lo, hi, tot)                                                       \
  if (blockIdx.x == 0) {                                                          \
    const int n_ = atomicAdd(&g_pprof_n, 0);                                      \
    if (n_ < 64) {                                                                \
      g_pprof[n_][tot] = clock64() - _start;                                      \
      for (int i_ = lo; i_ < hi; ++i_) g_pprof[n_][i_] = _acc[i_];                \
    }                                                                             \
  }
#else
#define PT0() ((void)0)
#define PTADD(i) ((void)0)
#define PTDECL() ((void)0)
#define PTSAVE(lo, hi, tot) ((void)0)
#endif

constexpr int kWarps = 18;
constexpr int kThreads = 32 * kWarps;
constexpr int kProdWarp = 0, kMmaWarp = 1, kEpiWarp0 = 2;
constexpr int kEpiWarps = 16;

template <bool SILU>
__device__ __forceinline__ float act_p(float x, int a) {
  if constexpr (SILU) return a == 2 ? __fdividef(x, 1.f + __expf(-x)) : (a ? fmaxf(x, 0.f) : x);
  else return a ? fmaxf(x, 0.f) : x;
}

__device__ __forceinline__ int atom_steps(const PairTerm& T, int a) {   // K=16 steps of atom a
  return min(T.aw / 16, (T.R - a * T.aw + 15) / 16);
}

template <bool SILU>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kThreads, 1)
    pair_chain_kernel(const __grid_constant__ PairDesc d, RunPtrs p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  const int S = d.stages, NB = d.nbuf;
  uint8_t* ring = smem;
  uint8_t* pbuf = smem + S * kSlot;
  float* sbias = reinterpret_cast<float*>(pbuf + kPBytes);
  uint64_t* bars = reinterpret_cast<uint64_t*>(pbuf + kPBytes + d.bias_bytes);
  uint64_t* full = bars;               // [S]  leader: producer expect_tx + both CTAs' TMA bytes
  uint64_t* empty = bars + S;          // [S]  each CTA: MMA commit (multicast)
  uint64_t* acc_full = bars + 2 * S;   // [NB] each CTA: level accumulator written (multicast)
  uint64_t* acc_empty = acc_full + 4;  // [NB] leader: 32 epilogue warps loaded it
  uint64_t* p_full = acc_empty + 4;    //      leader: 32 warps wrote P
  uint64_t* p_empty = p_full + 1;      //      each CTA: fconv MMAs read P (multicast)
  uint64_t* out_full = p_empty + 1;    //      each CTA: out accumulated (multicast)
  uint64_t* out_empty = out_full + 1;  //      leader: 32 warps drained out
  uint32_t* tslot = reinterpret_cast<uint32_t*>(out_empty + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t cta = cluster_ctarank();
  // per-unit atom program (identical for every unit): the producer and the issuer walk it
  // from shared memory instead of re-reading term fields from the (constant-cached) params
  uint2* prog = reinterpret_cast<uint2*>(bars) + 64;   // after the barriers, <= 64 entries
  if (warp == kProdWarp && lane == 0) {
    int n = 0, j = 0;
    for (int l = 0; l < d.n_levels; ++l) {
      const int n0 = n;
      for (; j < d.lvl_end[l]; ++j) {
        const PairTerm& T = d.term[j];
        for (int a = 0; a < T.natoms; ++a, ++n)
          prog[n] = make_uint2((uint32_t)j | ((uint32_t)T.aw << 8) | ((uint32_t)atom_steps(T, a) << 16) |
                                   ((n == n0 ? 1u : 0u) << 24) | ((l == 0 ? 4u : 0u) << 24),
                               (uint32_t)(a * T.aw));
      }
      prog[n - 1].x |= 2u << 24;   // last atom of the level
    }
    prog[n - 1].x |= 8u << 24;     // last atom of the unit
  }
  if (warp == kProdWarp && lane == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < 4; ++i) {
      mbar_init(&acc_full[i], 1);
      mbar_init(&acc_empty[i], 2 * kEpiWarps);
    }
    mbar_init(p_full, 2 * kEpiWarps);
    mbar_init(p_empty, 1);
    mbar_init(out_full, 1);
    mbar_init(out_empty, 2 * kEpiWarps);
    fence_mbar_init_cluster();
    for (int j = 0; j < d.n_terms; ++j) {
      prefetch_tmap(d.term[j].amap);
      prefetch_tmap(d.term[j].wmap);
    }
    prefetch_tmap(d.fmap);
  }
  if (warp >= kEpiWarp0) {
    const float4* src = reinterpret_cast<const float4*>(p.params + d.lbias);
    float4* dst = reinterpret_cast<float4*>(sbias);
    for (int i = threadIdx.x - 32 * kEpiWarp0; i < d.n_levels * d.Cpad / 4; i += 32 * kEpiWarps) dst[i] = __ldg(src + i);
  }
  if (warp == kMmaWarp) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  tc_fence_before();
  cluster_sync_all();
  tc_fence_after();
  const uint32_t tbase = *tslot;
  const uint32_t tout = tbase + (uint32_t)(NB * kPairWu);   // out region
  pdl_wait();

  const int pair_id = blockIdx.x >> 1, npairs = gridDim.x >> 1;
  const int U = d.nunits, D = d.n_levels;

  if (warp == kProdWarp) {
    // ------------------------------------------------------------ TMA producer (both CTAs)
    if (lane == 0) {
      int stage = 0;
      uint32_t ph = 0;
#ifdef TEMCO_TRACE
      const bool notma = (g_pdbg & 1) != 0;
#else
      constexpr bool notma = false;
#endif
      auto acquire = [&](uint32_t bytes) -> uint32_t {   // next ring stage; returns the leader's full barrier
        mbar_wait(&empty[stage], ph ^ 1);
        if (cta == 0) mbar_expect_tx(&full[stage], notma ? 0u : bytes);
        return mapa_shared(smem_u32(&full[stage]), 0);
      };
      auto next = [&]() {
        if (++stage == S) stage = 0, ph ^= 1;
      };
      auto fconv_atoms = [&](int u) {   // F[:, u*128 + a*64 .. +64], this CTA's Np/2 rows
        for (int a = 0; a < kPairWu / 64; ++a) {
          const uint32_t fb = acquire(2u * (uint32_t)(d.Np / 2 * 64 * 2));
          if (!notma) tma_load_2d_pair(ring + stage * kSlot, d.fmap, fb, u * kPairWu + a * 64, (int)cta * (d.Np / 2));
          next();
        }
      };
      int pend = -1;   // unit whose fconv follows the next work item's first level
      const uint8_t* term0 = reinterpret_cast<const uint8_t*>(&d.term[0]);
      for (int tile = pair_id; tile < d.ntiles; tile += npairs) {
        const int row0 = tile * 256 + (int)cta * 128;
        for (int u = 0; u < U; ++u) {
          for (int k = 0;; ++k) {
            const uint2 op = prog[k];
            const int j = op.x & 0xFF, aw = (op.x >> 8) & 0xFF;
            const uint32_t fl = op.x >> 24;
            const PairTerm* T = reinterpret_cast<const PairTerm*>(term0 + j * sizeof(PairTerm));
            const uint32_t fb = acquire(2u * (uint32_t)((128 + 64) * aw * 2));   // both CTAs, A + B
            uint8_t* sa = ring + stage * kSlot;
            if (!notma) {
              tma_load_2d_pair(sa, T->amap, fb, (int)op.y, row0);
              tma_load_2d_pair(sa + kSlotA, T->wmap, fb, (int)op.y, u * kPairWu + (int)cta * 64);
            }
            next();
            if ((fl & 6u) == 6u && pend >= 0) {   // after level 0: the previous unit's fconv operands
              fconv_atoms(pend);
              pend = -1;
            }
            if (fl & 8u) break;
          }
          pend = u;
        }
      }
      if (pend >= 0) fconv_atoms(pend);
    }
  } else if (warp == kMmaWarp) {
    // ------------------------------------------------------------ MMA issuer (leader, whole warp)
    if (cta == 0) {
      PTDECL();
      const uint32_t idesc_t = idesc_bf16(256, kPairWu), idesc_f = idesc_bf16(256, d.Np);
      const uint32_t sbase = smem_u32(smem), pbase = smem_u32(pbuf);
      int stage = 0;
      uint32_t ph = 0;
      int gl = 0;        // levels issued (accumulator buffer gl % NB, use gl / NB)
      int nf = 0;        // fconvs issued (P phase)
      int it = 0;        // tiles whose out region was started
      auto fconv = [&](int u) {
        PT0();
        mbar_wait_cluster(p_full, (uint32_t)nf & 1u);
        PTADD(3);
        tc_fence_after();
        if (u == 0 && it > 0) {   // a new tile's out region: previous tile drained
          PT0();
          mbar_wait_cluster(out_empty, (uint32_t)(it - 1) & 1u);
          PTADD(4);
          tc_fence_after();
        }
        for (int a = 0; a < kPairWu / 64; ++a) {
          PT0();
          mbar_wait(&full[stage], ph);
          PTADD(1);
          tc_fence_after();
          const uint64_t fd = umma_desc_k(sbase + stage * kSlot, 64);
          const uint64_t pd = umma_desc_k(pbase + a * 16384, 64);
          for (int k = 0; k < 4; ++k)
            mma2_bf16_w(tout, pd + 2 * k, fd + 2 * k, idesc_f, (u == 0 && a == 0 && k == 0) ? 0u : 1u);
          mma2_commit_mc_w(&empty[stage], 3);
          if (++stage == S) stage = 0, ph ^= 1;
        }
        mma2_commit_mc_w(p_empty, 3);
        ++nf;
        if (u == U - 1) {
          mma2_commit_mc_w(out_full, 3);
          ++it;
        }
      };
      int pend = -1;
      int b = 0, bu = 0;   // accumulator buffer of the current level, its use count
      for (int tile = pair_id; tile < d.ntiles; tile += npairs) {
        for (int u = 0; u < U; ++u) {
          uint32_t dt = 0;
          for (int k = 0;; ++k) {
            const uint2 op = prog[k];
            const int aw = (op.x >> 8) & 0xFF, nk = (op.x >> 16) & 0xFF;
            const uint32_t fl = op.x >> 24;
            if (fl & 1u) {   // first atom of a level: its buffer must have been drained
              if (bu > 0) {
                PT0();
                mbar_wait_cluster(&acc_empty[b], (uint32_t)(bu - 1) & 1u);
                PTADD(2);
                tc_fence_after();
              }
              dt = tbase + (uint32_t)(b * kPairWu);
            }
            PT0();
            mbar_wait(&full[stage], ph);
            PTADD(1);
            tc_fence_after();
            const uint32_t sa = sbase + stage * kSlot;
            const uint64_t ad = umma_desc_k(sa, aw), bd = umma_desc_k(sa + kSlotA, aw);
            PT0();
            for (int kk = 0; kk < nk; ++kk)
              mma2_bf16_w(dt, ad + 2 * kk, bd + 2 * kk, idesc_t, ((fl & 1u) && kk == 0) ? 0u : 1u);
            PTADD(5);
            PT0();
            mma2_commit_mc_w(&empty[stage], 3);
            PTADD(6);
            if (++stage == S) stage = 0, ph ^= 1;
            if (fl & 2u) {   // last atom of the level
              mma2_commit_mc_w(&acc_full[b], 3);
              if (++b == NB) b = 0, ++bu;
              if ((fl & 4u) && pend >= 0) {
                fconv(pend);
                pend = -1;
              }
            }
            if (fl & 8u) break;
          }
          pend = u;
        }
      }
      if (pend >= 0) fconv(pend);
      if (lane == 0) PTSAVE(1, 8, 0);
    }
  } else {
    // ------------------------------------------------------------ epilogue (16 warps, both CTAs)
    const int q = warp & 3;                  // TMEM lane quarter of this warp
    const int g = (warp - kEpiWarp0) >> 2;   // 32-column group of a unit
    const int row = q * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    const uint32_t pfull_c = mapa_shared(smem_u32(p_full), 0);
    const uint32_t oempty_c = mapa_shared(smem_u32(out_empty), 0);
    __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(const_cast<void*>(loc_ptr(d.y, p)));
    int b = 0, br = 0, np = 0, it = 0;   // accumulator buffer, its round
    PTDECL();
    for (int tile = pair_id; tile < d.ntiles; tile += npairs, ++it) {
      const int64_t prow = (int64_t)tile * 256 + cta * 128 + row;
      for (int u = 0; u < U; ++u) {
        float t[32];
        for (int l = 0; l < D; ++l) {
          const int act = d.act[l];
          const float4* b4 = reinterpret_cast<const float4*>(sbias + l * d.Cpad + u * kPairWu + g * 32);
          PT0();
          mbar_wait(&acc_full[b], (uint32_t)br & 1u);
          PTADD(9);
          tc_fence_after();
          uint32_t v[32];
          PT0();
          tmem_ld32(tbase + lane_off + (uint32_t)(b * kPairWu + g * 32), v);
          tmem_wait_ld();
          tc_fence_before();
          warp_arrive_cluster(mapa_shared(smem_u32(&acc_empty[b]), 0));
          if (++b == NB) b = 0, ++br;
          PTADD(11);
          PT0();
#pragma unroll
          for (int i4 = 0; i4 < 8; ++i4) {
            const float4 bb = b4[i4];   // broadcast LDS.128
            const float bq[4] = {bb.x, bb.y, bb.z, bb.w};
#pragma unroll
            for (int k = 0; k < 4; ++k) {
              const int i = 4 * i4 + k;
              const float z = __uint_as_float(v[i]) + bq[k];
              t[i] = act_p<SILU>(l == 0 ? z : z + t[i], act);
            }
          }
          PTADD(12);
        }
        // P = bf16(t_D) for the unit's fconv
        PT0();
        if (np > 0) mbar_wait(p_empty, (uint32_t)(np - 1) & 1u);
        PTADD(10);
        PT0();
        ++np;
        uint8_t* P = pbuf + (g >> 1) * 16384 + row * 128;
#pragma unroll
        for (int c4 = 0; c4 < 4; ++c4) {
          uint4 pk;
          pk.x = pack_bf16(t[8 * c4 + 0], t[8 * c4 + 1]);
          pk.y = pack_bf16(t[8 * c4 + 2], t[8 * c4 + 3]);
          pk.z = pack_bf16(t[8 * c4 + 4], t[8 * c4 + 5]);
          pk.w = pack_bf16(t[8 * c4 + 6], t[8 * c4 + 7]);
          const int chunk = (g & 1) * 4 + c4;
          *reinterpret_cast<uint4*>(P + ((chunk ^ (row & 7)) * 16)) = pk;
        }
        fence_proxy_async();
        warp_arrive_cluster(pfull_c);
        PTADD(14);
      }
      // out tile: TMEM columns [128 NB, 128 NB + Np) -> bf16 -> y[prow, :Nout]
      PT0();
      mbar_wait(out_full, (uint32_t)it & 1u);
      PTADD(13);
      PT0();
      tc_fence_after();
      const int nch = d.Np / 8;
      for (int c8 = g; c8 < nch; c8 += 4) {
        uint32_t v[8];
        tmem_ld8(tout + lane_off + c8 * 8, v);
        tmem_wait_ld();
        if (prow < d.npix && c8 * 8 < d.Nout) {
          uint4 pk;
          pk.x = pack_bf16(__uint_as_float(v[0]), __uint_as_float(v[1]));
          pk.y = pack_bf16(__uint_as_float(v[2]), __uint_as_float(v[3]));
          pk.z = pack_bf16(__uint_as_float(v[4]), __uint_as_float(v[5]));
          pk.w = pack_bf16(__uint_as_float(v[6]), __uint_as_float(v[7]));
          *reinterpret_cast<uint4*>(y + prow * d.Nout + c8 * 8) = pk;
        }
      }
      tc_fence_before();
      warp_arrive_cluster(oempty_c);
      PTADD(15);
    }
    if (warp == kEpiWarp0 && lane == 0) PTSAVE(9, 16, 8);
  }
  tc_fence_before();
  cluster_sync_all();
  if (warp == kMmaWarp) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(tbase));
  }
#ifdef TEMCO_TRACE
  if (blockIdx.x == 0 && threadIdx.x == 0) atomicAdd(&g_pprof_n, 1);
#endif
}

}  // namespace

void launch_pair_chain(const PairDesc& d, const RunPtrs& p, cudaStream_t s) {
  static int nsm = 0;
  if (!nsm) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    if (nsm < 2) nsm = 2;
  }
  const int npairs = std::min(nsm / 2, d.ntiles);
  if (d.silu) {
    static bool attr = false;
    if (!attr) {
      cudaFuncSetAttribute(pair_chain_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
      attr = true;
    }
    launch_pdl(pair_chain_kernel<true>, dim3(2 * npairs), dim3(kThreads), d.smem_bytes, s, d, p);
  } else {
    static bool attr = false;
    if (!attr) {
      cudaFuncSetAttribute(pair_chain_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
      attr = true;
    }
    launch_pdl(pair_chain_kernel<false>, dim3(2 * npairs), dim3(kThreads), d.smem_bytes, s, d, p);
  }
}

}  // namespace pair
}  // namespace temco


#ifdef TEMCO_TRACE
extern "C" int temco_debug_pair_prof(unsigned long long* out) {
  int n = 0;
  cudaMemcpyFromSymbol(&n, temco::pair::g_pprof_n, sizeof(int));
  cudaMemcpyFromSymbol(out, temco::pair::g_pprof, sizeof(unsigned long long) * 64 * 16);
  const int z = 0;
  cudaMemcpyToSymbol(temco::pair::g_pprof_n, &z, sizeof(int));
  return n;
}
extern "C" void temco_debug_pair_dbg(int v) { cudaMemcpyToSymbol(temco::pair::g_pdbg, &v, sizeof(int)); }
#endif
