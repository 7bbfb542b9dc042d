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
// Warp roles (18 warps): 0-15 epilogue (both CTAs), 16 TMA producer (both), 17 TMEM
// allocator (both) and MMA issuer (leader CTA).  Barriers the issuer waits on
// live in the leader CTA (peer arrivals through shared::cluster addresses);
// commits are multicast to both CTAs.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cmath>
#include <cstring>
#include <set>

#include "tmap.h"
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
constexpr int kSlotB = 8192;             // 64 rows x 64 bf16: this CTA's half of one unit's Lhat atom
constexpr int kSlotC = 2048;             // 64 rows x 16 bf16 (bias-MMA groups: this CTA's half of a level bias atom)
// ring stage: A + B for both units of a pair (+ C for both with bias-MMA): PairDesc::slot bytes
constexpr int kOnesBytes = 4096;         // 128 rows x 16 bf16 "ones" A tile of the bias MMA
constexpr int kPBytes = 128 * kPairWu * 2;   // P of one unit: two SW128 atoms of 128 x 64
constexpr int kBarBytes = 1024 + 16 * kPairMaxAtoms;   // barriers (first 1 KB) + the issuer's atom table (kTabOff)
constexpr int kTabOff = 1024;
constexpr int kPairMaxStages = 16;
constexpr int kChunk = 2;                // ring stages of one level consumed per (u0 pass, u1 pass)

}  // namespace

bool pair_lower_chain(const IR& ir, const Step& s, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                      std::vector<float>& params, PairDesc& d) {
  if (getenv("TEMCO_NO_PAIR")) return false;
  // roots: the fconv, or every fconv of a merged group (reading R37), all reading the same t
  std::vector<int> roots = {s.out};
  roots.insert(roots.end(), s.extra.begin(), s.extra.end());
  if ((int)roots.size() > kPairMaxOuts) return false;
  const int tsrc = ir.oin[s.out][0];
  int Nout = 0;
  for (int r : roots) {
    const Node& rn = ir.nodes[r];
    if (rn.role != ROLE_FCONV || rn.b || ir.oin[r].size() != 1 || ir.oin[r][0] != tsrc) return false;   // no bias (O1)
    if (rn.C % 8) return false;
    Nout += rn.C;
  }
  const Node& tn = ir.nodes[tsrc];
  const int C = tn.C;
  if (Nout % 8 || (Nout + 15) / 16 * 16 > 256) return false;
  ChainParser P{ir, std::set<int>(s.members.begin(), s.members.end()), C, {}, tn.H, tn.W};
  P.allow_silu = true;
  P.allow_member_act = true;
  for (int r : roots) P.members.erase(r);
  std::vector<PLevel> levels;
  if (!P.chain(tsrc, levels)) return false;
  if (P.visited != P.members) return false;
  int nterms = 0;
  for (auto& L : levels) {
    if (!L.pm.empty()) return false;
    for (auto& t : L.terms) {
      if (t.tk != 1) return false;   // plain terms (a concat member covers its channel range only)
      const int r = ir.oin[t.lconv][0];
      const Loc& l = loc.at(r);
      const Node& rn = ir.nodes[r];
      if (l.where != W_ARENA || l.dtype != DT_BF16 || rn.C % 8 || rn.H != tn.H || rn.W != tn.W) return false;
      ++nterms;
    }
  }
  if ((int)levels.size() > kPairMaxLevels || nterms > kPairMaxTerms || nterms == 0) return false;
  for (int r : roots) {
    const Loc& yl = loc.at(r);
    if (yl.where != W_ARENA || yl.dtype != DT_BF16) return false;
  }

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
  d.n_out = (int)roots.size();
  d.ycol[0] = 0;
  for (int k = 0; k < d.n_out; ++k) {
    d.ys[k] = loc.at(roots[k]);
    d.ycol[k + 1] = d.ycol[k] + ir.nodes[roots[k]].C;
  }
  d.n_levels = (int)levels.size();
  {
    const char* e = getenv("TEMCO_PAIR_FCONV_LAG");
    d.flag = std::min(d.n_levels - 1, e ? atoi(e) : 0);
  }
  int64_t flops = 0, bytes = 0;
  while (params.size() % 4) params.push_back(0.f);
  d.lbias = (int64_t)params.size();
  d.ngroups = d.Cpad / 32;
  for (int l = 0; l < d.n_levels; ++l) {
    const PLevel& L = levels[l];
    d.act[l] = L.relu ? 1 : L.silu ? 2 : 0;
    d.silu |= L.silu ? 1 : 0;
    for (int c = 0; c < d.Cpad; ++c) params.push_back(c < C ? (float)L.bias[c] : 0.f);
    if (!L.act_ch.empty()) {   // activated concat members: one activation per 32-channel group
      if (d.n_levels * d.ngroups > kPairMaxActGroups) return false;
      d.mixed_act = 1;
    }
    for (int gi = 0; gi < d.ngroups; ++gi) {
      int a = -2;
      for (int c = gi * 32; c < std::min(C, gi * 32 + 32); ++c) {
        const int ac = L.act_ch.empty() || L.act_ch[c] < 0 ? d.act[l] : L.act_ch[c];
        if (a == -2) a = ac;
        else if (a != ac) return false;   // an activation boundary inside a 32-channel group
        if (ac == 2) d.silu = 1;
      }
      if (l * d.ngroups + gi < kPairMaxActGroups) d.actg[l * d.ngroups + gi] = (uint8_t)(a < 0 ? 0 : a);
    }
  }
  int j = 0;
  std::vector<int> term_c0, term_c1;   // restored channel range of each term
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
      std::vector<float> w((size_t)d.Cpad * T.Rw, 0.f);   // rows outside [c0, c0 + C_term) stay zero
      for (int c = 0; c < lc.C; ++c)
        for (int k = 0; k < R; ++k) w[(size_t)(t.c0 + c) * T.Rw + k] = (float)(t.scale[c] * (*lc.w)[(size_t)c * R + k]);
      T.w = push_bf16(tcw, w);
      term_c0.push_back(t.c0);
      term_c1.push_back(t.c0 + lc.C);
      flops += d.npix * 2LL * lc.C * R;
      bytes += d.npix * 2LL * R;
    }
    d.lvl_end[l] = j;
  }
  d.n_terms = j;
  // per-unit-pair atom programs, in the launch parameters: pair pp runs the atoms of the terms
  // whose restored channel range meets its 256 channels (every term of a residual chain; a
  // concat member only in the pair(s) holding its channels -- DenseNet's 32-channel members)
  {
    const int UPn = (d.nunits + 1) / 2;
    if (UPn > kPairMaxUnitPairs) return false;
    int n = 0;
    for (int pp = 0; pp < UPn; ++pp) {
      d.pstart[pp] = (int16_t)n;
      const int ch0 = pp * 2 * kPairWu, ch1 = std::min(C, ch0 + 2 * kPairWu);
      for (int l = 0, jj = 0; l < d.n_levels; ++l) {
        const int n0 = n;
        for (; jj < d.lvl_end[l]; ++jj) {
          if (term_c1[jj] <= ch0 || term_c0[jj] >= ch1) continue;
          const PairTerm& T = d.term[jj];
          for (int a = 0; a < T.natoms; ++a, ++n) {
            if (n >= kPairMaxAtoms) return false;
            const int nk = std::min(T.aw / 16, (T.R - a * T.aw + 15) / 16);
            d.prog[n][0] = (uint32_t)jj | ((uint32_t)T.aw << 8) | ((uint32_t)nk << 16) | ((n == n0 ? 1u : 0u) << 24) |
                           ((l == 0 ? 4u : 0u) << 24) | ((uint32_t)l << 28);
            d.prog[n][1] = (uint32_t)(a * T.aw);
          }
        }
        if (n == n0) return false;      // a level with nothing in this pair (not produced by the parser)
        d.prog[n - 1][0] |= 2u << 24;   // last atom of the level
      }
      d.prog[n - 1][0] |= 8u << 24;     // last atom of the pair's program
    }
    d.n_prog = n;
  }
  std::vector<float> f((size_t)d.Np * d.Cpad, 0.f);   // the roots' F stacked row-wise
  for (int k = 0; k < d.n_out; ++k) {
    const Node& rn = ir.nodes[roots[k]];
    for (int o = 0; o < rn.C; ++o)
      for (int c = 0; c < C; ++c) f[(size_t)(d.ycol[k] + o) * d.Cpad + c] = (*rn.w)[(size_t)o * C + c];
  }
  d.F = push_bf16(tcw, f);
  d.alg_flops = flops + d.npix * 2LL * Nout * C;
  d.alg_bytes = bytes + d.npix * 2LL * Nout;
  // small-rank groups (every level K <= 64: the epilogue, not the tensor core, bounds them)
  // add the level bias through the tensor core: one K=16 MMA of a constant ones tile times
  // [hi(b), lo(b)] bf16 columns (error ~2^-16 |b|), so the epilogue does no bias work
  {
    int kmax = 0;
    for (int l = 0, jj = 0; l < d.n_levels; ++l) {
      int k = 0;
      for (; jj < d.lvl_end[l]; ++jj) k += d.term[jj].R;
      kmax = std::max(kmax, k);
    }
    d.bias_mma = getenv("TEMCO_PAIR_NO_BIASMMA") ? 0 : 1;
  }
  if (d.bias_mma) {
    std::vector<float> bm((size_t)d.n_levels * d.Cpad * 16, 0.f);
    for (int l = 0; l < d.n_levels; ++l)
      for (int c = 0; c < C; ++c) {
        const float x = (float)levels[l].bias[c];
        uint32_t u;
        memcpy(&u, &x, 4);
        u &= 0xFFFF0000u;   // hi: truncated to bf16 exactly; lo = remainder (rounded to bf16 at upload)
        float hi;
        memcpy(&hi, &u, 4);
        bm[((size_t)l * d.Cpad + c) * 16 + 0] = hi;
        bm[((size_t)l * d.Cpad + c) * 16 + 1] = x - hi;
      }
    d.bmat = push_bf16(tcw, bm);
  }
  // level biases live in shared memory (fp32 [n_levels][Cpad]): L1 is ~empty next to
  // 200+ KB of shared memory, so per-level global bias loads would each cost an L2 trip
  d.bias_bytes = (d.n_levels * d.Cpad * 4 + 1023) / 1024 * 1024;
  if (d.bias_mma) d.bias_bytes = 0;
  d.nbuf = std::min(3, (512 - d.Np) / kPairWu);   // 3 for Np <= 128, 2 for Np <= 256
  const int budget = 227 * 1024 - 1024 /*align*/ - kBarBytes - 2 * kPBytes - d.bias_bytes - kOnesBytes;
  // resident weights: per unit pair pp and program atom k, this CTA's halves of both units'
  // Lhat atoms; per (pp, level) the bias-MMA atoms; per (unit, 64-channel atom) F
  {
    int awmax = 16;
    for (int jj = 0; jj < d.n_terms; ++jj) awmax = std::max(awmax, (int)d.term[jj].aw);
    const int UP = (d.nunits + 1) / 2;
    d.bsz = 64 * awmax * 2;
    d.fsz = d.Np / 2 * 128;
    const int rb = d.n_prog * 2 * d.bsz;
    const int rc = d.bias_mma ? UP * d.n_levels * 2 * kSlotC : 0;
    const int rf = d.nunits * 2 * d.fsz;
    d.res_c = (rb + 1023) / 1024 * 1024;
    d.res_f = d.res_c + (rc + 1023) / 1024 * 1024;
    d.res_bytes = d.res_f + (rf + 1023) / 1024 * 1024;
    int64_t tx = 0;
    for (int pp = 0; pp < UP; ++pp) {
      const int nu = std::min(2, d.nunits - 2 * pp);
      const int pend = pp + 1 < UP ? d.pstart[pp + 1] : d.n_prog;
      for (int k = d.pstart[pp]; k < pend; ++k) tx += nu * 64 * (int)((d.prog[k][0] >> 8) & 0xFF) * 2;
      if (d.bias_mma) tx += (int64_t)nu * d.n_levels * 64 * 16 * 2;
    }
    tx += (int64_t)d.nunits * 2 * d.fsz;
    d.res_tx = (int)tx;
    const int slot_r = 128 * awmax * 2;
    const int st_r = std::min(kPairMaxStages, (budget - d.res_bytes) / slot_r);
    int maxp = 0;   // longest unit-pair program
    for (int pp = 0; pp < UP; ++pp) maxp = std::max(maxp, (pp + 1 < UP ? d.pstart[pp + 1] : d.n_prog) - d.pstart[pp]);
    d.resident = !getenv("TEMCO_PAIR_NO_RES") && st_r >= std::max(8, maxp + 2) ? 1 : 0;
    if (d.resident) {
      d.slot = slot_r;
      d.stages = st_r;
    }
  }
  if (!d.resident) {
    d.res_bytes = 0;
    // ring stages sized by the widest K atom of the group (an r atom of 128 rows, both units' Lhat
    // halves of 64 rows, the bias atoms) and by one fconv F atom (Np/2 rows of 64 columns): rank-8
    // concat members (DenseNet) take 12 KB stages, so 16 of them are in flight instead of 4 x 36 KB
    int awmax = 16;
    for (int jj = 0; jj < d.n_terms; ++jj) awmax = std::max(awmax, (int)d.term[jj].aw);
    d.sa = 128 * awmax * 2;
    d.sb = 64 * awmax * 2;
    d.slot = std::max(d.sa + 2 * d.sb + (d.bias_mma ? 2 * kSlotC : 0), d.Np / 2 * 128);
    d.slot = (d.slot + 1023) / 1024 * 1024;
    const char* e = getenv("TEMCO_PAIR_FIXED_SLOTS");
    if (e && atoi(e)) {
      d.sa = kSlotA;
      d.sb = kSlotB;
      d.slot = kSlotA + 2 * kSlotB + (d.bias_mma ? 2 * kSlotC : 0);
    }
    d.stages = std::min(e && atoi(e) ? 8 : kPairMaxStages, budget / d.slot);
  }
  if (d.stages < 2 * kChunk) return false;
  d.smem_bytes = 1024 + d.res_bytes + d.stages * d.slot + 2 * kPBytes + d.bias_bytes + kOnesBytes + kBarBytes;
  return true;
}

bool pair_finalize(size_t n, const std::function<PairDesc*(size_t)>& get, char* arena, uint16_t* tcw,
                   std::string& err) {
  bool any = false;
  for (size_t i = 0; i < n; ++i) any |= get(i) != nullptr;
  if (!any) return true;
  const auto encode = tmap_encoder(err);
  if (!encode) return false;
  auto make = [&](unsigned char* dst, void* base, uint64_t inner, uint64_t outer, uint32_t box_outer, int aw) {
    return tmap_2d_bf16(encode, dst, base, inner, outer, (uint32_t)aw, box_outer, tmap_swizzle_bf16(aw));
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
    if (d->bias_mma && !make(d->bmap, tcw + d->bmat, 16, (uint64_t)d->n_levels * d->Cpad, 64, 16)) {
      err = "cuTensorMapEncodeTiled failed (pair bias)";
      return false;
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
// experiment builds only: event timeline of CTA 0 (rows: see scripts/pair_timeline.py)
__device__ long long g_ev[16][512];
__device__ int g_ev_on, g_launch;
__device__ int g_pdbg;   // timing experiments: 1 = producer issues no TMA, 2 = epilogue skips TMEM / math
#define EVDECL() int _evn[16] = {0}; const bool _evon = blockIdx.x == 0 && g_launch == g_ev_on
#define EV(row)                                                                                   \
  do {                                                                                            \
    if (_evon && _evn[row] < 512) g_ev[row][_evn[row]++] = clock64();                             \
  } while (0)
#else
#define EVDECL() ((void)0)
#define EV(row) ((void)0)
#endif

// epilogue waits: sleep on the barrier (suspend-time hint) rather than re-issuing
// try_wait, so 16 waiting warps do not take issue slots from the producer / issuer
#ifdef TEMCO_PAIR_SPIN
#define PAIR_EPI_WAIT(b, p) mbar_wait(b, p)
#else
#define PAIR_EPI_WAIT(b, p) mbar_wait_sleep(b, p)
#endif

constexpr int kWarps = 18;
constexpr int kThreads = 32 * kWarps;
// epilogue warps first: the SM sub-partition arbiter favours the highest warp id, so the
// single-thread producer and MMA issuer (warps 16, 17) win issue slots over the 16
// epilogue warps sharing their sub-partitions
constexpr int kEpiWarp0 = 0, kProdWarp = 16, kMmaWarp = 17;
constexpr int kEpiWarps = 16;

__device__ __forceinline__ void add2(float& a0, float& a1, float b0, float b1) {   // packed FADD2
  asm("{\n.reg .b64 x, y;\nmov.b64 x, {%0, %1};\nmov.b64 y, {%2, %3};\nadd.rn.f32x2 x, x, y;\nmov.b64 {%0, %1}, x;\n}\n"
      : "+f"(a0), "+f"(a1)
      : "f"(b0), "f"(b1));
}

__device__ __forceinline__ uint32_t pack_relu(float lo, float hi) {   // bf16x2(max(lo, 0), max(hi, 0))
  uint32_t r;
  asm("cvt.rn.relu.bf16x2.f32 %0, %2, %1;" : "=r"(r) : "f"(lo), "f"(hi));
  return r;
}

template <bool SILU>
__device__ __forceinline__ float silu_or(float x, int act) {
  if constexpr (SILU) return act == 2 ? silu_fast(x) : x;
  else return x;
}

// One level of one unit for this thread's 32 channels: t (bf16x2, 16 words) =
// act(a (+ bias) (+ t)), a = the level accumulator from TMEM (fp32).  t is held in
// bf16 between levels -- the precision the unfused bf16 model stores every
// intermediate tensor in -- and each level rounds once.
template <bool SILU>
__device__ __forceinline__ void level_math(uint32_t (&t)[16], const uint32_t (&v)[32], bool first, int act,
                                           const float* bias) {
  if (!bias && act != 2) {
    // bias added by the tensor core (bias MMA): t = act(a + t) in packed bf16x2 -- the level
    // accumulator a rounded to bf16 (cvt, one instruction per two channels), then one fused
    // a * 1 + t with the ReLU (fma.rn.relu.bf16x2) rounding once: two instructions per two
    // channels instead of unpacking t to fp32 (reading R29: t lives in bf16 between levels)
    if (first) {
#pragma unroll
      for (int i = 0; i < 16; ++i)
        t[i] = act == 1 ? pack_relu(__uint_as_float(v[2 * i]), __uint_as_float(v[2 * i + 1]))
                        : pack_bf16(__uint_as_float(v[2 * i]), __uint_as_float(v[2 * i + 1]));
    } else if (act == 1) {
#pragma unroll
      for (int i = 0; i < 16; ++i) {
        const uint32_t a2 = pack_bf16(__uint_as_float(v[2 * i]), __uint_as_float(v[2 * i + 1]));
        asm("fma.rn.relu.bf16x2 %0, %1, %2, %0;" : "+r"(t[i]) : "r"(a2), "r"(0x3F803F80u));
      }
    } else {
#pragma unroll
      for (int i = 0; i < 16; ++i) {
        const uint32_t a2 = pack_bf16(__uint_as_float(v[2 * i]), __uint_as_float(v[2 * i + 1]));
        asm("fma.rn.bf16x2 %0, %1, %2, %0;" : "+r"(t[i]) : "r"(a2), "r"(0x3F803F80u));
      }
    }
    return;
  }
  float z[32];
#pragma unroll
  for (int i = 0; i < 32; ++i) z[i] = __uint_as_float(v[i]);
  if (bias) {
    const float4* b4 = reinterpret_cast<const float4*>(bias);
#pragma unroll
    for (int i4 = 0; i4 < 8; ++i4) {
      const float4 bb = b4[i4];   // broadcast LDS.128
      add2(z[4 * i4], z[4 * i4 + 1], bb.x, bb.y);
      add2(z[4 * i4 + 2], z[4 * i4 + 3], bb.z, bb.w);
    }
  }
  if (!first) {
#pragma unroll
    for (int i = 0; i < 16; ++i) add2(z[2 * i], z[2 * i + 1], __uint_as_float(t[i] << 16), __uint_as_float(t[i] & 0xFFFF0000u));
  }
  if (act == 1) {
#pragma unroll
    for (int i = 0; i < 16; ++i) t[i] = pack_relu(z[2 * i], z[2 * i + 1]);
  } else if (SILU && act == 2) {
#pragma unroll
    for (int i = 0; i < 16; ++i) t[i] = pack_silu_bf16(z[2 * i], z[2 * i + 1]);
  } else {
#pragma unroll
    for (int i = 0; i < 16; ++i) t[i] = pack_bf16(silu_or<SILU>(z[2 * i], act), silu_or<SILU>(z[2 * i + 1], act));
  }
}

template <bool SILU>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kThreads, 1)
    pair_chain_kernel(const __grid_constant__ PairDesc d, RunPtrs p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  const int S = d.stages, kSlot = d.slot;
  uint8_t* res = smem;                                              // resident weights (d.resident)
  uint8_t* ring = smem + d.res_bytes;
  uint8_t* pbuf = ring + S * kSlot;                                 // P of unit 0 | unit 1 of a pair
  uint8_t* ones = pbuf + 2 * kPBytes;                               // bias-MMA A tile (1024-aligned)
  float* sbias = reinterpret_cast<float*>(ones + kOnesBytes);
  uint64_t* bars = reinterpret_cast<uint64_t*>(ones + kOnesBytes + d.bias_bytes);
  uint64_t* full = bars;               // [S]  leader: producer expect_tx + both CTAs' TMA bytes
  uint64_t* empty = bars + 16;         // [S]  each CTA: MMA commit (multicast)
  uint64_t* acc_full = bars + 32;      // [NB] each CTA: a (unit, level) accumulator written (multicast)
  uint64_t* acc_empty = bars + 36;     // [NB] leader: 32 epilogue warps loaded it
  uint64_t* p_full = bars + 40;        //      leader: 32 warps wrote P of both units
  uint64_t* p_empty = bars + 41;       //      each CTA: fconv MMAs read P (multicast)
  uint64_t* out_full = bars + 42;      //      each CTA: out accumulated (multicast)
  uint64_t* out_empty = bars + 43;     //      leader: 32 warps drained out
  uint64_t* wbar = bars + 44;          //      leader: resident weights landed (both CTAs' bytes)
  uint32_t* tslot = reinterpret_cast<uint32_t*>(bars + 45);
  const int NB = d.nbuf;               // rotating 128-column accumulators: item i -> buffer i % NB
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t cta = cluster_ctarank();
  if (warp == kProdWarp && lane == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < NB; ++i) {
      mbar_init(&acc_full[i], 1);
      mbar_init(&acc_empty[i], 2 * kEpiWarps);
    }
    mbar_init(p_full, 2 * kEpiWarps);
    mbar_init(p_empty, 1);
    mbar_init(out_full, 1);
    mbar_init(out_empty, 2 * kEpiWarps);
    mbar_init(wbar, 1);
    fence_mbar_init_cluster();
    for (int jj = 0; jj < d.n_terms; ++jj) {
      prefetch_tmap(d.term[jj].amap);
      prefetch_tmap(d.term[jj].wmap);
    }
    prefetch_tmap(d.fmap);
    if (d.bias_mma) prefetch_tmap(d.bmap);
  }
  if (warp < kEpiWarp0 + kEpiWarps) {
    if (d.bias_mma) {
      // ones tile, K-major SW32 (32-byte rows; 16-byte chunk c of row r at c ^ ((r >> 2) & 1)):
      // K columns 0 and 1 = 1.0 (they meet the bias hi / lo columns), the rest 0
      const int r = threadIdx.x - 32 * kEpiWarp0;
      if (r < 128) {
        uint4* rowp = reinterpret_cast<uint4*>(ones + r * 32);
        const int c0 = (r >> 2) & 1;
        rowp[c0] = make_uint4(0x3F803F80u, 0u, 0u, 0u);
        rowp[c0 ^ 1] = make_uint4(0u, 0u, 0u, 0u);
      }
      fence_proxy_async();
    } else {
      const float4* src = reinterpret_cast<const float4*>(p.params + d.lbias);
      float4* dst = reinterpret_cast<float4*>(sbias);
      for (int i = threadIdx.x - 32 * kEpiWarp0; i < d.n_levels * d.Cpad / 4; i += 32 * kEpiWarps) dst[i] = __ldg(src + i);
    }
  }
  if (warp == kMmaWarp) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  tc_fence_before();
  cluster_sync_all();
  tc_fence_after();
  // the CTA allocates all 512 TMEM columns, so the base address is lane 0 / column 0: a
  // compile-time constant keeps the issuer's accumulator addresses in uniform registers
  if (*tslot != 0u) __trap();
  constexpr uint32_t tbase = 0;
  const uint32_t tout = tbase + (uint32_t)(NB * kPairWu);   // out region [128 NB, 128 NB + Np)
  pdl_wait();

  const int pair_id = blockIdx.x >> 1, npairs = gridDim.x >> 1;
  const int U = d.nunits, UP = (U + 1) / 2;   // 128-channel units, unit pairs

  if (warp == kProdWarp) {
    // ------------------------------------------------------------ TMA producer (both CTAs)
    if (lane == 0) {
      int stage = 0;
      uint32_t ph = 0;
// next ring stage (waits until the MMAs freed it); fb = the leader's full barrier of the stage
#ifdef TEMCO_TRACE
      const bool notma = (g_pdbg & 1) != 0;
#else
      constexpr bool notma = false;
#endif
#define PAIR_ACQUIRE(bytes)                                            \
  mbar_wait(&empty[stage], ph ^ 1);                                    \
  if (cta == 0) mbar_expect_tx(&full[stage], notma ? 0u : (bytes));    \
  const uint32_t fb = mapa_shared(smem_u32(&full[stage]), 0)
#define PAIR_NEXT()           \
  if (++stage == S) {         \
    stage = 0;                \
    ph ^= 1;                  \
  }
#define PAIR_FCONV_ATOMS(pp)                                                                                   \
  for (int u = 2 * (pp); u < min(2 * (pp) + 2, U); ++u)                                                        \
    for (int a = 0; a < kPairWu / 64; ++a) {                                                                   \
      PAIR_ACQUIRE(2u * (uint32_t)(d.Np / 2 * 64 * 2));                                                        \
      if (!notma) tma_load_2d_pair(ring + stage * kSlot, d.fmap, fb, u * kPairWu + a * 64, (int)cta * (d.Np / 2)); \
      PAIR_NEXT();                                                                                             \
    }
      EVDECL();
      int pend = -1;   // pair whose fconv operands follow the next pair's first level
      const uint8_t* term0 = reinterpret_cast<const uint8_t*>(&d.term[0]);
      if (d.resident) {   // every weight atom of this CTA's halves, once
        if (cta == 0) mbar_expect_tx(wbar, 2u * (uint32_t)d.res_tx);
        const uint32_t wb = mapa_shared(smem_u32(wbar), 0);
        for (int pp = 0; pp < UP; ++pp) {
          const int u0 = 2 * pp, nu = min(2, U - u0);
          const int pend = pp + 1 < UP ? d.pstart[pp + 1] : d.n_prog;
          for (int k = d.pstart[pp]; k < pend; ++k) {
            const uint2 op = make_uint2(d.prog[k][0], d.prog[k][1]);
            const PairTerm* T = reinterpret_cast<const PairTerm*>(term0 + (op.x & 0xFF) * sizeof(PairTerm));
            for (int q = 0; q < nu; ++q) {
              tma_load_2d_pair(res + (k * 2 + q) * d.bsz, T->wmap, wb, (int)op.y,
                               (u0 + q) * kPairWu + (int)cta * 64);
              if (d.bias_mma && ((op.x >> 24) & 1u))
                tma_load_2d_pair(res + d.res_c + ((pp * d.n_levels + (int)(op.x >> 28)) * 2 + q) * kSlotC, d.bmap, wb, 0,
                                 (int)(op.x >> 28) * d.Cpad + (u0 + q) * kPairWu + (int)cta * 64);
            }
          }
        }
        for (int u = 0; u < U; ++u)
          for (int a = 0; a < kPairWu / 64; ++a)
            tma_load_2d_pair(res + d.res_f + (u * 2 + a) * d.fsz, d.fmap, wb, u * kPairWu + a * 64, (int)cta * (d.Np / 2));
      }
      for (int tile = pair_id; tile < d.ntiles; tile += npairs) {
        const int row0 = tile * 256 + (int)cta * 128;
        for (int pp = 0; pp < UP; ++pp) {
          const int u0 = 2 * pp, nu = min(2, U - u0);
          for (int k = d.pstart[pp];; ++k) {
            const uint2 op = make_uint2(d.prog[k][0], d.prog[k][1]);
            const int j = op.x & 0xFF, aw = (op.x >> 8) & 0xFF;
            const uint32_t fl = op.x >> 24;
            const PairTerm* T = reinterpret_cast<const PairTerm*>(term0 + j * sizeof(PairTerm));
            const bool bia = d.bias_mma && (fl & 1u) && !d.resident;
            PAIR_ACQUIRE(2u * (uint32_t)((128 + (d.resident ? 0 : 64 * nu)) * aw * 2 + (bia ? nu * 64 * 32 : 0)));
            uint8_t* sa = ring + stage * kSlot;
            EV(0);
            if (!notma) tma_load_2d_pair(sa, T->amap, fb, (int)op.y, row0);
            for (int q = 0; q < nu && !notma && !d.resident; ++q) {
              tma_load_2d_pair(sa + d.sa + q * d.sb, T->wmap, fb, (int)op.y, (u0 + q) * kPairWu + (int)cta * 64);
              if (bia)
                tma_load_2d_pair(sa + d.sa + 2 * d.sb + q * kSlotC, d.bmap, fb, 0,
                                 (int)(op.x >> 28) * d.Cpad + (u0 + q) * kPairWu + (int)cta * 64);
            }
            PAIR_NEXT();
            if ((fl & 2u) && (int)(op.x >> 28) == d.flag && pend >= 0 && !d.resident) {   // after level flag: the previous pair's fconv operands
              PAIR_FCONV_ATOMS(pend);
              pend = -1;
            }
            if (fl & 8u) break;
          }
          pend = pp;
        }
      }
      if (pend >= 0 && !d.resident) {
        PAIR_FCONV_ATOMS(pend);
      }
#undef PAIR_ACQUIRE
#undef PAIR_NEXT
#undef PAIR_FCONV_ATOMS
    }
  } else if (warp == kMmaWarp) {
    // ------------------------------------------------------------ MMA issuer (leader, whole warp;
    // one elected lane issues each tcgen05 instruction)
    if (cta == 0) {
      const uint32_t idesc_t = idesc_bf16(256, kPairWu), idesc_f = idesc_bf16(256, d.Np);
      const uint32_t rbase = smem_u32(res), sbase = smem_u32(ring), pbase = smem_u32(pbuf);
      // per-atom table (shared memory; the param-space program would be a dynamically indexed
      // constant load per atom): {program word, descriptor hi of its K atom width, resident
      // Lhat descriptor lo (pair 0, unit 0), resident bias descriptor lo (pair 0, unit 0)}
      uint4* tab = reinterpret_cast<uint4*>(reinterpret_cast<uint8_t*>(bars) + kTabOff);
      for (int k = lane; k < d.n_prog; k += 32) {
        const uint32_t x = d.prog[k][0];
        const int aw = (x >> 8) & 0xFF;
        tab[k] = make_uint4(x, udesc_hi(aw), udesc_lo(rbase + (uint32_t)(k * 2 * d.bsz)),
                            udesc_lo(rbase + (uint32_t)(d.res_c + (int)(x >> 28) * 2 * kSlotC)));
      }
      __syncwarp();
      const uint32_t tab_s = smem_u32(tab);
      if (d.resident) {
        mbar_wait_u(wbar, 0);
        tc_fence_after();
      }
      const uint32_t a_lo0 = udesc_lo(sbase), slot16 = (uint32_t)kSlot >> 4;
      const uint32_t hi16 = udesc_hi(16), hi64 = udesc_hi(64), ones_lo = udesc_lo(smem_u32(ones));
      const uint32_t bq16 = (uint32_t)d.bsz >> 4;
      const uint32_t pc_step = (uint32_t)(d.n_levels * 2 * kSlotC) >> 4, cq16 = (uint32_t)kSlotC >> 4;
      int stage = 0;
      uint32_t ph = 0;
      int b = 0;                   // accumulator buffer of the next item (items rotate over NB)
      uint32_t used = 0, par = 0;  // per buffer: used before / parity of its next acc_empty wait
      int nf = 0;                  // pair fconvs issued
      int it = 0;                  // tiles whose out region was started
// fconv of unit pair pp: out (+)= P_u F_u^T for its units; the first pair of a tile starts
// the out region (after the previous tile's out was drained), the last one publishes it
#define PAIR_FCONV(pp, first_of_tile, last_of_tile)                                                            \
  {                                                                                                            \
    EV(14);                                                                                                    \
    mbar_wait_u(p_full, (uint32_t)nf & 1u);                                                                    \
    EV(4);                                                                                                     \
    tc_fence_after();                                                                                          \
    if ((first_of_tile) && it > 0) {                                                                           \
      mbar_wait_u(out_empty, (uint32_t)(it - 1) & 1u);                                                         \
      tc_fence_after();                                                                                        \
    }                                                                                                          \
    for (int q = 0; q < min(2, U - 2 * (pp)); ++q) {                                                           \
      if (d.resident) {   /* both 64-channel F atoms of unit q: one block of 8 MMAs */                         \
        mma2_k8_w(tout, udesc_lo(pbase + (uint32_t)(q * kPBytes)), hi64,                                       \
                  udesc_lo(rbase + (uint32_t)(d.res_f + (2 * (pp) + q) * 2 * d.fsz)), hi64, 16384u,             \
                  (uint32_t)d.fsz, idesc_f, ((first_of_tile) && q == 0) ? 0u : 1u);                            \
      } else {                                                                                                 \
        for (int a = 0; a < kPairWu / 64; ++a) {                                                               \
          mbar_wait_u(&full[stage], ph);                                                                       \
          tc_fence_after();                                                                                    \
          mma2_k4_w(tout, udesc_lo(pbase + (uint32_t)(q * kPBytes + a * 16384)), hi64,                         \
                    a_lo0 + (uint32_t)stage * slot16, hi64, idesc_f,                                           \
                    ((first_of_tile) && q == 0 && a == 0) ? 0u : 1u, 4u);                                      \
          mma2_commit_mc_w(&empty[stage], 3);                                                                  \
          if (++stage == S) stage = 0, ph ^= 1;                                                                \
        }                                                                                                      \
      }                                                                                                        \
    }                                                                                                          \
    mma2_commit_mc_w(p_empty, 3);                                                                              \
    EV(15);                                                                                                    \
    ++nf;                                                                                                      \
    if (last_of_tile) {                                                                                        \
      mma2_commit_mc_w(out_full, 3);                                                                           \
      ++it;                                                                                                    \
    }                                                                                                          \
  }
      EVDECL();
      int pend = -1, pend_tile_first = 0, pend_tile_last = 0;
      for (int tile = pair_id; tile < d.ntiles; tile += npairs) {
        for (int pp = 0; pp < UP; ++pp) {
          const int nu = min(2, U - 2 * pp);
          const uint32_t pco = (uint32_t)pp * pc_step;
          int k = d.pstart[pp];
          for (;;) {   // one level per iteration, in chunks of <= kChunk ring stages
            const uint32_t op0x = lds128(tab_s + 16u * k).x;
            int kl = k;   // last atom of this level
            while (!((lds128(tab_s + 16u * kl).x >> 24) & 2u)) ++kl;
            const int nat = kl - k + 1;
            int b1 = b + 1;   // buffer of the pair's second unit
            if (b1 >= NB) b1 -= NB;
            const uint32_t d0 = tbase + (uint32_t)(b * kPairWu), d1 = tbase + (uint32_t)(b1 * kPairWu);
            for (int c0 = 0; c0 < nat; c0 += kChunk) {
              const int cn = min(kChunk, nat - c0);
              if (c0 == 0) {   // new items in buffers b (, b1): their previous items must have been drained
                for (int q = 0; q < nu; ++q) {
                  const int bq = q ? b1 : b;
                  if ((used >> bq) & 1u) {
#ifdef TEMCO_TRACE
                    if (!(g_pdbg & 4)) {   // timing experiment 4: no acc_empty waits
#endif
                    EV(12);
                    mbar_wait_u(&acc_empty[bq], (par >> bq) & 1u);
                    EV(13);
#ifdef TEMCO_TRACE
                    }
#endif
                    par ^= 1u << bq;
                  } else {
                    used |= 1u << bq;
                  }
                }
                tc_fence_after();
              }
              int st = stage;
              uint32_t sph = ph;
              for (int i = 0; i < cn; ++i) {
                const uint4 tk = lds128(tab_s + 16u * (k + c0 + i));
                mbar_wait_u(&full[st], sph);
                EV(1);
                tc_fence_after();
                const bool lvl0 = c0 == 0 && i == 0;   // first atom of the level
                const bool bia = d.bias_mma && lvl0;
                const uint32_t a_lo = a_lo0 + (uint32_t)st * slot16;
                const uint32_t b0_lo = d.resident ? tk.z : a_lo + ((uint32_t)d.sa >> 4);
                const uint32_t b1_lo = b0_lo + (d.resident ? bq16 : ((uint32_t)d.sb >> 4));
                const uint32_t c0_lo = d.resident ? tk.w + pco : a_lo + ((uint32_t)(d.sa + 2 * d.sb) >> 4);
                const uint32_t c1_lo = c0_lo + (d.resident ? cq16 : ((uint32_t)kSlotC >> 4));
                mma2_atom2_w(d0, d1, a_lo, tk.y, b0_lo, b1_lo, c0_lo, c1_lo, ones_lo, hi16, idesc_t, (tk.x >> 16) & 0xFFu,
                             (uint32_t)nu, bia ? 1u : 0u, (lvl0 && !bia) ? 0u : 1u);
                EV(2);
                if (++st == S) st = 0, sph ^= 1;
              }
              if (c0 + cn == nat) {
                mma2_commit2_mc_w(smem_u32(&acc_full[b]), smem_u32(&acc_full[b1]), (uint32_t)nu);
                EV(3);
              }
              {   // release the chunk's ring stages (kChunk = 2: one block)
                int s1 = stage + 1;
                if (s1 == S) s1 = 0;
                mma2_commit2_mc_w(smem_u32(&empty[stage]), smem_u32(&empty[s1]), (uint32_t)cn);
                for (int i = 0; i < cn; ++i)
                  if (++stage == S) stage = 0, ph ^= 1;
              }
            }
            b += nu;
            if (b >= NB) b -= NB;
            if ((int)(op0x >> 28) == d.flag && pend >= 0) {   // the previous pair's fconv, d.flag levels late
              PAIR_FCONV(pend, pend_tile_first, pend_tile_last);
              pend = -1;
            }
            const bool last = (lds128(tab_s + 16u * kl).x >> 24) & 8u;
            k = kl + 1;
            if (last) break;
          }
          pend = pp;
          pend_tile_first = pp == 0;
          pend_tile_last = pp == UP - 1;
        }
      }
      if (pend >= 0) PAIR_FCONV(pend, pend_tile_first, pend_tile_last);
#undef PAIR_FCONV
    }
  } else {
    // ------------------------------------------------------------ epilogue (16 warps, both CTAs)
    const int q = warp & 3;                  // TMEM lane quarter of this warp (warp % 4)
    const int g = (warp - kEpiWarp0) >> 2;   // 32-column group of a unit
    const int row = q * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    const uint32_t pfull_c = mapa_shared(smem_u32(p_full), 0);
    const uint32_t oempty_c = mapa_shared(smem_u32(out_empty), 0);

    int gi = 0, np = 0, it = 0;   // gi: (unit, level) accumulator items consumed
    int eb = 0;                   // buffer of item gi (gi mod NB)
    uint32_t ephase = 0;          // per buffer: parity of its next acc_full phase
    const uint32_t aempty_c = mapa_shared(smem_u32(&acc_empty[0]), 0);   // leader's acc_empty[0]
    EVDECL();
    const bool ev0 = warp == kEpiWarp0 && lane == 0;
    // out tile of tile `oit` (pixel row orow): TMEM columns [128 NB, 128 NB + Np) -> bf16 -> y.
    // The issuer runs a tile's last fconv after the NEXT tile's level 0, so the epilogue
    // drains that out region after consuming the next tile's level-0 items (not before
    // them: that would idle the epilogue for a whole fconv round trip per tile)
    auto drain_out = [&](int oit, int64_t orow) {
      PAIR_EPI_WAIT(out_full, (uint32_t)oit & 1u);
      tc_fence_after();
      const int nch = d.Np / 8;
      for (int c8 = g; c8 < nch; c8 += 4) {
        uint32_t v[8];
        tmem_ld8(tout + lane_off + c8 * 8, v);
        tmem_wait_ld();
        if (orow < d.npix && c8 * 8 < d.Nout) {
          uint4 pk;
          pk.x = pack_bf16(__uint_as_float(v[0]), __uint_as_float(v[1]));
          pk.y = pack_bf16(__uint_as_float(v[2]), __uint_as_float(v[3]));
          pk.z = pack_bf16(__uint_as_float(v[4]), __uint_as_float(v[5]));
          pk.w = pack_bf16(__uint_as_float(v[6]), __uint_as_float(v[7]));
          int k = 0;   // output holding column c8 * 8 (a merged group's fconvs, reading R37)
          while (k + 1 < d.n_out && c8 * 8 >= d.ycol[k + 1]) ++k;
          __nv_bfloat16* yk = reinterpret_cast<__nv_bfloat16*>(const_cast<void*>(loc_ptr(d.ys[k], p)));
          *reinterpret_cast<uint4*>(yk + orow * (d.ycol[k + 1] - d.ycol[k]) + (c8 * 8 - d.ycol[k])) = pk;
        }
      }
      tc_fence_before();
      warp_arrive_cluster(oempty_c);
      if (ev0) EV(11);
    };
    int pend_it = -1;
    int64_t pend_row = 0;
    for (int tile = pair_id; tile < d.ntiles; tile += npairs, ++it) {
      const int64_t prow = (int64_t)tile * 256 + cta * 128 + row;
      for (int pp = 0; pp < UP; ++pp) {
        const int nu = min(2, U - 2 * pp);
        uint32_t t0[16], t1[16];
        for (int l = 0; l < d.n_levels; ++l) {
#pragma unroll
          for (int qq = 0; qq < 2; ++qq) {
            if (qq < nu) {
              const int act = d.mixed_act ? (int)d.actg[l * d.ngroups + (2 * pp + qq) * (kPairWu / 32) + g] : d.act[l];
              const float* bl = d.bias_mma ? nullptr : sbias + l * d.Cpad + (2 * pp + qq) * kPairWu + g * 32;
              // item gi + qq: buffer (gi + qq) mod NB and its use parity, kept incrementally (no division)
              int b = eb + qq;
              if (b >= NB) b -= NB;
              PAIR_EPI_WAIT(&acc_full[b], (ephase >> b) & 1u);
              ephase ^= 1u << b;
              if (ev0) EV(qq ? 8 : 5);
              tc_fence_after();
              uint32_t v[32];
#ifdef TEMCO_TRACE
              if (g_pdbg & 2) {
                warp_arrive_cluster(mapa_shared(smem_u32(&acc_empty[b]), 0));
                continue;
              }
#endif
              tmem_ld32(tbase + lane_off + (uint32_t)(b * kPairWu + g * 32), v);
              tmem_wait_ld();
              tc_fence_before();
              warp_arrive_cluster(aempty_c + 8u * (uint32_t)b);
              if (ev0 && !qq) EV(6);
              level_math<SILU>(qq ? t1 : t0, v, l == 0, act, bl);
              if (ev0) EV(qq ? 9 : 7);
            }
          }
          gi += nu;
          eb += nu;
          if (eb >= NB) eb -= NB;
          if (l == d.flag && pp == 0 && pend_it >= 0) {
            drain_out(pend_it, pend_row);
            pend_it = -1;
          }
        }
        // P = t_D (already bf16x2) of both units for the pair's fconv
        if (np > 0) PAIR_EPI_WAIT(p_empty, (uint32_t)(np - 1) & 1u);
        ++np;
#pragma unroll
        for (int qq = 0; qq < 2; ++qq) {
          if (qq < nu) {
            uint8_t* P = pbuf + qq * kPBytes + (g >> 1) * 16384 + row * 128;
            const uint32_t* t = qq ? t1 : t0;
#pragma unroll
            for (int c4 = 0; c4 < 4; ++c4) {
              const int chunk = (g & 1) * 4 + c4;
              *reinterpret_cast<uint4*>(P + ((chunk ^ (row & 7)) * 16)) =
                  make_uint4(t[4 * c4], t[4 * c4 + 1], t[4 * c4 + 2], t[4 * c4 + 3]);
            }
          }
        }
        fence_proxy_async();
        warp_arrive_cluster(pfull_c);
        if (ev0) EV(10);
      }
      pend_it = it;
      pend_row = prow;
    }
    if (pend_it >= 0) drain_out(pend_it, pend_row);
  }
  tc_fence_before();
  cluster_sync_all();
  if (warp == kMmaWarp) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(tbase));
  }
#ifdef TEMCO_TRACE
  if (blockIdx.x == 0 && threadIdx.x == 0) g_launch = g_launch + 1;
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
// timeline of CTA 0 for the tc_pair launch with index `launch` (counted from the last reset)
extern "C" void temco_debug_pair_ev(int launch, long long* out) {
  if (out) cudaMemcpyFromSymbol(out, temco::pair::g_ev, sizeof(long long) * 16 * 512);
  cudaMemcpyToSymbol(temco::pair::g_ev_on, &launch, sizeof(int));
  const int z = 0;
  cudaMemcpyToSymbol(temco::pair::g_launch, &z, sizeof(int));
  static long long zz[16 * 512] = {0};
  cudaMemcpyToSymbol(temco::pair::g_ev, zz, sizeof(zz));
}
extern "C" void temco_debug_pair_dbg(int v) { cudaMemcpyToSymbol(temco::pair::g_pdbg, &v, sizeof(int)); }
#endif
