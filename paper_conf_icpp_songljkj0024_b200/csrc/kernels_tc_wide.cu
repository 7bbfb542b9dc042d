// tcgen05 fused restore-chain kernel, wide-group variant (sm_100a): the level
// value accumulates in TMEM (ReLU pass via tcgen05.st between levels), 128-channel
// units in pairs.  Chosen for groups whose reduced inputs of one tile do not fit
// in shared memory (kernels_tc.cu keeps them resident and t in registers).
//
// One fused group computes, per output tile,
//     t_l = act_l( sum_{j in l} r_j Lhat_j^T + b_l + t_{l-1} ),  out = t_D F^T
// with the C-wide t never leaving the SM:
//   GEMM1  r_j atoms [rows x 64] (2D TMA of 128 consecutive pixels, or 4D TMA of
//          a tap-shifted, strided spatial box) and Lhat_j atoms [Cc x 64] (TMA)
//          -> SMEM ring -> tcgen05.mma (M=128, N=Cc, K=16) -> TMEM accumulator;
//          the level bias enters the same accumulator through the tensor core
//          (constant SMEM ones tile x [b_hi, b_lo] columns)
//   level epilogue (8 warps: TMEM lane quarter x column half): TMEM -> regs,
//          ReLU, -> TMEM (tcgen05.st) so the next level accumulates on top of
//          t_{l-1}; after the last level the bf16 tile P = t_D goes to SMEM in
//          the SW128 K-major layout.  Pooled-member chunks keep one TMEM region
//          per tap and fold max / sum in registers; GAP roots reduce per image.
//   GEMM2  tcgen05.mma (A = P from SMEM, B = F atom via TMA) -> TMEM (Np columns)
//   output epilogue: TMEM -> registers -> bf16 -> global.
// Warp roles (320 threads, persistent over tiles): warps 0-7 epilogue, 8 TMA
// producer, 9 MMA issuer.  Units (a chunk, or a tap group of a pooled chunk)
// alternate between two TMEM buffers so one unit's MMAs overlap the previous
// unit's epilogue.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cmath>
#include <set>

#include "tmap.h"
#include "chain_lower.h"
#include "chain_parse.h"
#include "tc_wide.h"
#include "tc_ptx.cuh"

namespace temco {
namespace wide {

// ===========================================================================
// host: lowering
// ===========================================================================
namespace {
using namespace chainp;
using chainl::push_bf16;
using chainl::push_f32;
using chainl::to_bf16;


float from_bf16(uint16_t h) {
  uint32_t u = (uint32_t)h << 16;
  float f;
  memcpy(&f, &u, 4);
  return f;
}



// bias as a rank-2 term: columns 0, 1 = bf16 hi / lo parts (error ~2^-16 |b|)
int64_t push_bias(std::vector<uint16_t>& pool, const std::vector<double>& b, int c0, int Cpad) {
  std::vector<float> bm((size_t)Cpad * 8, 0.f);
  for (size_t c = 0; c < b.size(); ++c) {
    const float x = (float)b[c];
    const float hi = from_bf16(to_bf16(x));
    bm[(size_t)(c0 + c) * 8 + 0] = hi;
    bm[(size_t)(c0 + c) * 8 + 1] = x - hi;
  }
  return push_bf16(pool, bm);
}

// Per-tile producer / MMA programs.  Unit order (all roles): for each pair of
// units: for each level: for each unit of the pair: [bias, terms x taps x K
// atoms]; then the fconv atoms of the pair's finished chunks.  TMEM buffer of
// unit u of a tile = (units before the tile + u) & 1.
void build_programs(TcChainDesc& d, std::vector<uint16_t>& tcw) {
  std::vector<TcProdOp> P;
  std::vector<TcMmaOp> M;
  const int Cc = d.Cc;
  const int U = d.npc * d.ntg + d.nchunks - d.npc;
  d.units = U;
  const bool res = d.resident != 0;
  const int rows_a = d.spatial ? d.tw * d.th * d.tn : 128;
  const int pbytes = 128 * Cc * 2;
  auto moff = [&](const unsigned char* m) {
    return (uint16_t)((reinterpret_cast<const char*>(m) - reinterpret_cast<const char*>(&d)) / 64);
  };
  struct HUnit {
    int c, tg, nt;
    bool pooled, last;
  };
  auto unit_at = [&](int u) {
    HUnit x;
    if (u < d.npc * d.ntg) {
      x.c = u / d.ntg;
      x.tg = u % d.ntg;
      x.nt = std::min(d.tpu, d.mtaps - x.tg * d.tpu);
      x.pooled = true;
      x.last = x.tg == d.ntg - 1;
    } else {
      x.c = d.npc + (u - d.npc * d.ntg);
      x.tg = 0;
      x.nt = 1;
      x.pooled = false;
      x.last = true;
    }
    return x;
  };
  for (int u0 = 0; u0 < U; u0 += 2) {
    const int nb = std::min(2, U - u0);
    for (int l = 0; l < d.n_levels; ++l)
      for (int bi = 0; bi < nb; ++bi) {
        const int u = u0 + bi;
        const HUnit un = unit_at(u);
        // level biases are added by the epilogue: the first MMA into each tap region
        // at level 0 overwrites (MF_ZERO); a region no term reaches gets a zero-init MMA
        const size_t m_first = M.size();
        std::vector<char> region_done(un.nt, 0);
        const int j0 = un.pooled ? d.mt0 : (l ? d.lvl_end[l - 1] : 0);
        const int j1 = un.pooled ? d.mt1 : d.lvl_end[l];
        for (int r = 0; r < un.nt; ++r)
          for (int j = j0; j < j1; ++j) {
            const TcTerm& t = d.term[j];
            if (!un.pooled && !(t.c0 < (un.c + 1) * Cc && t.c0 + t.C > un.c * Cc)) continue;
            const int ntap = un.pooled ? 1 : t.tk * t.tk;
            const int katoms = t.Rp / t.aw;
            for (int q = 0; q < ntap; ++q) {
              const int tap = un.pooled ? un.tg * d.tpu + r : q;
              const int kk = un.pooled ? d.mk : t.tk, pad = un.pooled ? d.mp : t.tp;
              const int step = d.k2 ? 2 : 1;   // K atoms per ring stage
              for (int ka = 0; ka < katoms; ka += step) {
                const int n2 = std::min(step, katoms - ka);
                auto nk_of = [&](int a) { return std::min(t.aw / 16, (t.R - a * t.aw + 15) / 16); };
                TcProdOp o{};
                o.kind = d.spatial ? PK_A4D : PK_A2D;
                o.ts = (uint8_t)t.ts;
                o.amap = moff(d.spatial ? t.tmap4 : t.tmap);
                o.ac = (int16_t)(ka * t.aw);
                o.dx = (int16_t)(tap % kk - pad);
                o.dy = (int16_t)(tap / kk - pad);
                o.bytes = (uint32_t)(n2 * (rows_a + (res ? 0 : Cc)) * t.aw * 2);
                o.n2 = (uint8_t)n2;
                o.aw = (uint8_t)t.aw;
                o.bstep64 = (uint16_t)(Cc * t.aw * 2 / 64);
                if (!res) {
                  o.kind |= PK_B;
                  o.bmap = moff(t.wmap);
                  o.bx = (int16_t)(ka * t.aw);
                  o.by = (int16_t)(un.c * Cc);
                }
                P.push_back(o);
                TcMmaOp m{};
                m.flags = MF_SW | MF_SA | MF_SD | (res ? MF_BRES : MF_SB);
                if (l == 0 && !region_done[r]) m.flags |= MF_ZERO;
                region_done[r] = 1;
                m.unit = (uint8_t)u;
                m.nk = (uint8_t)(nk_of(ka) + (n2 == 2 ? nk_of(ka + 1) : 0));
                if (n2 == 2) {
                  m.nk1 = (uint8_t)nk_of(ka);
                  m.a2 = (uint16_t)((rows_a * t.aw * 2) >> 4);
                  m.b2 = (uint16_t)((Cc * t.aw * 2) >> 4);
                }
                m.la = (uint8_t)t.aw;
                m.lb = (uint8_t)t.aw;
                m.tcol = (uint16_t)(r * Cc);
                if (res) m.boff = (uint32_t)(t.wres + ((un.c - t.cfirst) * katoms + ka) * Cc * t.aw * 2);
                M.push_back(m);
              }
            }
          }
        for (int r = 0; r < un.nt; ++r)
          if (l == 0 && !region_done[r]) {   // zero-init: ones tile x zero tile
            TcMmaOp m{};
            m.flags = MF_ONES | MF_BZERO | MF_ZERO;
            m.unit = (uint8_t)u;
            m.nk = 1;
            m.la = 16;
            m.lb = 16;
            m.tcol = (uint16_t)(r * Cc);
            M.push_back(m);
          }
        M[m_first].flags |= MF_ACC_WAIT;
        M.back().flags |= MF_ACC_COMMIT;
      }
    if (!d.gap)
      for (int bi = 0; bi < nb; ++bi) {
        const HUnit un = unit_at(u0 + bi);
        if (!un.last) continue;
        const int pb = un.c & 1;
        const int na = Cc / 64;
        // two F atoms per stage with two-atom stages, when they fit the stage's B region
        const int fstep = (d.k2 && na == 2 && (res || 2 * d.Np * 128 <= d.slot_b)) ? 2 : 1;
        for (int a = 0; a < na; a += fstep) {
          if (!res) {
            TcProdOp o{};
            o.kind = PK_B;
            o.bmap = moff(d.fmap);
            o.bx = (int16_t)(un.c * Cc + a * 64);
            o.by = 0;
            o.bytes = (uint32_t)(fstep * d.Np * 128);
            o.n2 = (uint8_t)fstep;
            o.aw = 64;
            o.bstep64 = (uint16_t)(d.Np * 128 / 64);
            P.push_back(o);
          }
          TcMmaOp m{};
          m.flags = MF_F | (a == 0 ? MF_P_WAIT : 0) | (a == 0 && un.c == 0 ? MF_OUT_WAIT | MF_ZERO : 0) |
                    (a + fstep >= na ? MF_P_COMMIT : 0) | (res ? MF_BRES : MF_SW | MF_SB | MF_SD);
          m.unit = (uint8_t)pb;
          m.nk = (uint8_t)(4 * fstep);
          if (fstep == 2) {
            m.nk1 = 4;
            m.a2 = (uint16_t)(16384 >> 4);
            m.b2 = (uint16_t)((d.Np * 128) >> 4);
          }
          m.la = 64;
          m.lb = 64;
          m.aoff = (uint32_t)(pb * pbytes + a * 16384);
          if (res) m.boff = (uint32_t)(d.fres + (un.c * na + a) * d.Np * 128);
          M.push_back(m);
        }
      }
  }
  if (!d.gap) M.back().flags |= MF_OUT_COMMIT;
  d.n_prod = (int32_t)P.size();
  d.n_mma = (int32_t)M.size();
  // programs live in SMEM (after the pooled slab) when they fit next to the ring
  const int pbytes_prog = (int)(P.size() * sizeof(TcProdOp) + M.size() * sizeof(TcMmaOpD));
  d.prog_smem = 0;
  const char* exp_env = getenv("TEMCO_TC_EXP");   // experiment switches (bit 0: programs in global memory)
  const int exp_bits = exp_env ? atoi(exp_env) : 0;
  if (pbytes_prog <= 32768 && !(exp_bits & 1)) {
    const int need = (pbytes_prog + 127) / 128 * 128;
    while (d.stages > 2 && d.smem_bytes + need > 227 * 1024)
      d.stages--, d.smem_bytes -= d.slot_a + d.slot_b;
    if (d.smem_bytes + need <= 227 * 1024) {
      d.prog_smem = need;
      d.smem_bytes += need;
    }
  }
  // pipelined MMA order (unit ops of tile t+1 before the fconv ops of tile t):
  // needs resident weights (the ring then carries only unit stages, consumed in
  // the same order) and a program of the form [unit ops][fconv ops]
  d.mma_head = 0;
  // and every TMEM buffer the head of tile t+1 waits for must be released by the
  // epilogue before it waits for tile t's output: one level, <= 2 units per tile
  if (res && !d.gap && d.n_levels == 1 && U <= 2) {
    int h = 0;
    while (h < (int)M.size() && !(M[h].flags & MF_F)) ++h;
    bool tail_f = true;
    for (size_t i = h; i < M.size(); ++i) tail_f &= (M[i].flags & MF_F) != 0;
    if (tail_f && h > 0 && h < (int)M.size()) d.mma_head = h;
  }
  while (tcw.size() % 512) tcw.push_back(0);
  // device MMA ops: descriptors relative to the aligned SMEM base (final layout)
  const int slot = d.slot_a + d.slot_b;
  const uint32_t ring_off = (uint32_t)d.wres_bytes;
  const uint32_t pbuf_off = ring_off + (uint32_t)(d.stages * slot);
  const uint32_t ones_off = pbuf_off + 2u * (uint32_t)pbytes;
  auto dtmpl = [](uint32_t off, int aw) {
    const uint64_t layout = aw == 64 ? 2 : aw == 32 ? 4 : 6;
    return (uint64_t)(off >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(16 * aw >> 4) << 32) | ((uint64_t)1 << 46) |
           (layout << 61);
  };
  auto idesc = [](int M_, int N_) {
    return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N_ >> 3) << 17) | ((uint32_t)(M_ >> 4) << 24);
  };
  std::vector<TcMmaOpD> MD(M.size());
  for (size_t i = 0; i < M.size(); ++i) {
    const TcMmaOp& m = M[i];
    TcMmaOpD& o = MD[i];
    const bool isF = m.flags & MF_F;
    const uint32_t aoff = (m.flags & MF_ONES) ? ones_off : isF ? pbuf_off + m.aoff : ring_off;
    const uint32_t boff = (m.flags & MF_BZERO) ? ones_off + 4096u : (m.flags & MF_BRES) ? m.boff : ring_off + (uint32_t)d.slot_a;
    o.adesc = dtmpl(aoff, m.la);
    o.bdesc = dtmpl(boff, m.lb);
    o.idesc = isF ? idesc(128, d.Np) : idesc(128, Cc);
    o.tmem = (isF ? (uint32_t)(2 * d.ubuf) : m.tcol) | ((uint32_t)m.nk1 << 24);
    o.flags = m.flags;
    o.unit = m.unit;
    o.nk = m.nk;
    o.a2 = m.a2;
    o.b2 = m.b2;
  }
  d.prog_off = (int64_t)tcw.size();
  const size_t nbytes = P.size() * sizeof(TcProdOp) + MD.size() * sizeof(TcMmaOpD);
  tcw.resize(tcw.size() + (nbytes + 1) / 2);
  char* dst = reinterpret_cast<char*>(tcw.data() + d.prog_off);
  memcpy(dst, P.data(), P.size() * sizeof(TcProdOp));
  memcpy(dst + P.size() * sizeof(TcProdOp), MD.data(), MD.size() * sizeof(TcMmaOpD));
}

}  // namespace

bool tc_lower_chain(const IR& ir, const Step& s, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                    std::vector<float>& params, TcChainDesc& d) {
  const Node& root = ir.nodes[s.out];
  const bool gap = root.op == OP_GAP;
  if (root.role != ROLE_FCONV && !gap) return false;
  if (!gap && root.b) return false;              // fconv factors carry no bias (O1)
  const int tsrc = ir.oin[s.out][0];
  const Node& tn = ir.nodes[tsrc];
  const int C = tn.C, Nout = gap ? 16 : root.C;
  if (Nout % 8 || Nout > 256) return false;
  if (gap && tn.H * tn.W > 128) return false;
  ChainParser P{ir, std::set<int>(s.members.begin(), s.members.end()), C, {}, tn.H, tn.W};
  P.allow_silu = true;
  P.members.erase(s.out);
  std::vector<PLevel> levels;
  if (!P.chain(tsrc, levels)) return false;
  if (P.visited != P.members) return false;          // every member must be part of the chain form
  // pooled members / tap-accumulate terms: single level, member in the leading channels
  bool taps_any = false;
  for (auto& L : levels)
    for (auto& t : L.terms) taps_any |= t.tk > 1;
  const PMember* pm = nullptr;
  for (auto& L : levels) {
    if (L.pm.size() > 1) return false;
    if (!L.pm.empty()) pm = &L.pm[0];
  }
  const bool mixed = pm || taps_any;
  if (mixed && levels.size() != 1) return false;
  if (pm && (pm->c0 != 0 || pm->C % 64)) return false;
  if (pm && gap) return false;                       // GAP over a max-pooled member: generic path
  int nterms = 0;
  for (auto& L : levels) nterms += (int)L.terms.size();
  if (pm) nterms += (int)pm->terms.size();
  if ((int)levels.size() > kTcMaxLevels || nterms > kTcMaxTerms) return false;
  auto term_ok = [&](const PTerm& t) {
    const int r = ir.oin[t.lconv][0];
    const Loc& l = loc.at(r);
    return l.where == W_ARENA && l.dtype == DT_BF16 && ir.nodes[r].C % 8 == 0;
  };
  for (auto& L : levels)
    for (auto& t : L.terms)
      if (!term_ok(t)) return false;
  if (pm)
    for (auto& t : pm->terms)
      if (!term_ok(t)) return false;
  const Loc& yl = loc.at(s.out);
  if (yl.where != W_ARENA || yl.dtype != DT_BF16) return false;

  d = TcChainDesc();
  d.C = C;
  d.Cc = (C <= 64 || mixed) ? 64 : 128;
  if (!chainl::tile_geometry(d, ir, tn, Nout, gap, mixed, yl, (int)levels.size())) return false;
  int64_t flops = 0, bytes = 0;
  int j = 0;
  auto add_term = [&](const PTerm& t) -> bool { return chainl::add_term(d, d.term[j++], ir, loc, tcw, t, flops, bytes); };
  for (int l = 0; l < d.n_levels; ++l) {
    const PLevel& L = levels[l];
    d.relu[l] = L.relu ? 1 : L.silu ? 2 : 0;
    // pooled-member channels take no level bias through the MMA: their level bias
    // (the post-BN shift) is added after pooling, in the epilogue
    std::vector<double> lb = L.bias;
    if (pm && l == 0) {
      std::vector<double> post(d.Cc * (pm->C / d.Cc), 0.0);
      for (int c = 0; c < pm->C; ++c) {
        post[c] = lb[c];
        lb[c] = 0.0;
      }
      while (params.size() % 4) params.push_back(0.f);
      d.post = (int64_t)params.size();
      for (double x : post) params.push_back((float)x);
      if (!pm->post_scale.empty()) {
        std::vector<double> ps(post.size(), 1.0);
        for (int c = 0; c < pm->C; ++c) ps[c] = pm->post_scale[c];
        while (params.size() % 4) params.push_back(0.f);
        d.postsc = (int64_t)params.size();
        for (double x : ps) params.push_back((float)x);
      }
    }
    d.boff[l] = push_bias(tcw, lb, 0, d.Cpad);
    d.lbias[l] = push_f32(params, lb, d.Cpad);
    for (const PTerm& t : L.terms)
      if (!add_term(t)) return false;
    d.lvl_end[l] = j;
  }
  d.n_terms = j;
  if (pm) {
    d.npc = pm->C / d.Cc;
    d.mpool = pm->kind;
    d.mk = pm->k;
    d.ms = pm->s;
    d.mp = pm->p;
    d.mtaps = pm->k * pm->k;
    d.mrelu = pm->relu ? 1 : pm->silu ? 2 : 0;
    d.mHin = pm->Hin;
    d.mWin = pm->Win;
    d.mt0 = j;
    for (const PTerm& t : pm->terms) {
      PTerm u = t;
      u.tk = 1;
      u.ts = pm->s;
      if (!add_term(u)) return false;
    }
    d.mt1 = j;
    // the member is evaluated once per tap: count its work at the taps actually run
    d.boffm = push_bias(tcw, pm->bias, 0, d.Cpad);
    d.mbias = push_f32(params, pm->bias, d.Cpad);
    if (d.tw * d.ms > 256 || d.th * d.ms > 256) return false;
  }
  d.F = 0;
  d.Fb = -1;
  if (gap) {
    d.alg_flops = flops + d.npix * C;
    d.alg_bytes = bytes + 2LL * ir.batch * C;
  } else {
    std::vector<float> f((size_t)d.Np * d.Cpad, 0.f);
    for (int o = 0; o < Nout; ++o)
      for (int c = 0; c < C; ++c) f[(size_t)o * d.Cpad + c] = (*root.w)[(size_t)o * C + c];
    d.F = push_bf16(tcw, f);
    d.alg_flops = flops + d.npix * 2LL * Nout * C;
    d.alg_bytes = bytes + d.npix * 2LL * Nout;
  }
  // pooled member: as many taps per unit as two unit buffers + the output allow
  d.tpu = 1;
  d.ntg = 1;
  if (pm) {
    int t = d.mtaps;
    while (t > 1 && 2 * t * d.Cc + d.Np > 512) --t;
    d.ntg = (d.mtaps + t - 1) / t;
    d.tpu = (d.mtaps + d.ntg - 1) / d.ntg;
  }
  d.ubuf = d.tpu * d.Cc;
  // shared memory: ring of (A | B) stages sized by the widest K atom of the group
  // (small ranks -> small stages -> a deep ring), two P tiles, ones tile, barriers
  int awmax = 16;
  const int nall = pm ? d.mt1 : d.n_terms;
  for (int i = 0; i < nall; ++i) awmax = std::max(awmax, d.term[i].aw);
  // two K atoms per ring stage when some term spans several atoms (ranks > 64: ResNet-50
  // stages 3-4): half the stages / commits / handshakes per MMA, measured -13..-26 % on those
  // groups (and +1-2 % on single-atom groups, which keep one atom per stage)
  int max_atoms = 1;
  for (int i = 0; i < (pm ? d.mt1 : d.n_terms); ++i) max_atoms = std::max(max_atoms, d.term[i].Rp / d.term[i].aw);
  d.k2 = (!pm && max_atoms >= 2 && !getenv("TEMCO_WIDE_NOK2")) ? 1 : 0;
  const int rows_a_l = d.spatial ? d.tw * d.th * d.tn : 128;
  d.slot_a = (d.k2 ? 2 : 1) * std::max(128, rows_a_l) * awmax * 2;
  int sb = std::max((d.k2 ? 2 : 1) * d.Cc * awmax * 2, d.Cc * 32);
  if (!gap) sb = std::max(sb, d.Np * 128);
  d.slot_b = (sb + 1023) / 1024 * 1024;
  const int pbytes = 128 * d.Cc * 2;
  const int runbytes = pm ? 32768 : 0;     // pooled member: running max / sum slab (after the barriers)
  const int budget = 227 * 1024 - 1024 /*align*/ - 2048 /*barriers*/ - runbytes - 2 * pbytes - 8192 /*ones, zeros*/;
  // resident weights: every B box (term atoms of the chunks a term reaches, level
  // and member biases, F atoms) once per CTA, if that leaves a ring of >= 6 A slots
  int64_t woff = 0;
  for (int i = 0; i < nall; ++i) {
    TcTerm& T = d.term[i];
    T.wres = (int32_t)woff;
    woff += (int64_t)T.nhit * (T.Rp / T.aw) * d.Cc * T.aw * 2;
  }
  d.fres = (int32_t)woff;
  if (!gap) woff += (int64_t)(d.Cpad / 64) * d.Np * 128;
  d.resident = woff + 6LL * d.slot_a <= budget ? 1 : 0;
  if (d.resident) {
    d.wres_bytes = (int32_t)woff;
    d.slot_b = 0;
    d.stages = std::min<int64_t>(24, (budget - woff) / d.slot_a);
  } else {
    d.wres_bytes = 0;
    d.stages = std::min(24, budget / (d.slot_a + d.slot_b));
  }
  if (d.stages < 2) return false;
  d.smem_bytes = 1024 + d.wres_bytes + d.stages * (d.slot_a + d.slot_b) + 2 * pbytes + 8192 + 2048 + runbytes;
  const int cols = 2 * d.ubuf + d.Np;
  d.tmem_cols = cols <= 32 ? 32 : cols <= 64 ? 64 : cols <= 128 ? 128 : cols <= 256 ? 256 : 512;
  if (cols > 512) return false;
  build_programs(d, tcw);
  return true;
}

bool tc_finalize(size_t n, const std::function<TcChainDesc*(size_t)>& get, char* arena, uint16_t* tcw,
                 std::string& err) {
  bool any = false;
  for (size_t i = 0; i < n; ++i) any |= get(i) != nullptr;
  if (!any) return true;
  const auto encode = tmap_encoder(err);
  if (!encode) return false;
  auto swz = [](int aw) { return tmap_swizzle_bf16(aw); };
  auto make = [&](unsigned char* dst, void* base, uint64_t inner, uint64_t outer, uint32_t box_outer, int aw = 64) {
    return tmap_2d_bf16(encode, dst, base, inner, outer, (uint32_t)aw, box_outer, swz(aw));
  };
  auto make4 = [&](unsigned char* dst, void* base, const TcChainDesc* d, const TcTerm& t) {
    cuuint64_t dims[4] = {(cuuint64_t)t.R, (cuuint64_t)t.Win, (cuuint64_t)t.Hin, (cuuint64_t)d->nimg};
    cuuint64_t strides[3] = {(cuuint64_t)t.R * 2, (cuuint64_t)t.Win * t.R * 2, (cuuint64_t)t.Hin * t.Win * t.R * 2};
    cuuint32_t box[4] = {(cuuint32_t)t.aw, (cuuint32_t)(d->tw * t.ts), (cuuint32_t)(d->th * t.ts), (cuuint32_t)d->tn};
    cuuint32_t es[4] = {1, (cuuint32_t)t.ts, (cuuint32_t)t.ts, 1};
    CUresult r = encode(reinterpret_cast<CUtensorMap*>(dst), CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, base, dims, strides,
                        box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, swz(t.aw),
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
  };
  for (size_t i = 0; i < n; ++i) {
    TcChainDesc* d = get(i);
    if (!d) continue;
    d->prod = reinterpret_cast<const TcProdOp*>(tcw + d->prog_off);
    d->mma = reinterpret_cast<const TcMmaOpD*>(reinterpret_cast<const char*>(d->prod) + d->n_prod * sizeof(TcProdOp));
    const int nt = d->npc ? d->mt1 : d->n_terms;
    for (int j = 0; j < nt; ++j) {
      TcTerm& t = d->term[j];
      bool ok = make(t.wmap, tcw + t.w, (uint64_t)t.Rw, (uint64_t)d->Cpad, (uint32_t)d->Cc, t.aw);
      if (d->spatial)
        ok = ok && make4(t.tmap4, arena + t.r.off, d, t);
      else
        ok = ok && make(t.tmap, arena + t.r.off, (uint64_t)t.R, (uint64_t)d->nimg * t.Hin * t.Win, 128, t.aw);
      if (!ok) {
        err = "cuTensorMapEncodeTiled failed (term)";
        return false;
      }
    }
    for (int l = 0; l < d->n_levels; ++l)
      if (!make(d->bmap[l], tcw + d->boff[l], 8, (uint64_t)d->Cpad, (uint32_t)d->Cc, 16)) {
        err = "cuTensorMapEncodeTiled failed (bias)";
        return false;
      }
    if (d->npc && !make(d->bmapm, tcw + d->boffm, 8, (uint64_t)d->Cpad, (uint32_t)d->Cc, 16)) {
      err = "cuTensorMapEncodeTiled failed (member bias)";
      return false;
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

// level activation: ReLU when a != 0; the SILU instantiation also takes a == 2 -> SiLU (
// fast approximate division, bf16 outputs).  ReLU-only plans launch SILU = false: epilogue unchanged
template <bool SILU>
__device__ __forceinline__ float act_w(float x, int a) {
  if constexpr (SILU) return a == 2 ? silu_fast(x) : (a ? fmaxf(x, 0.f) : x);
  else return a ? fmaxf(x, 0.f) : x;
}

__device__ __forceinline__ bool term_hits(const TcTerm& t, int c, int Cc) {
  return t.c0 < (c + 1) * Cc && t.c0 + t.C > c * Cc;
}

#ifdef TEMCO_TRACE
// experiment builds only: %globaltimer stamps of CTA 0's pipeline events
constexpr int kTraceRows = 12;
__device__ unsigned long long g_trace[kTraceRows][512];
__device__ int g_dbg;   // 1: TMA-only run (MMA / epilogue roles idle; output garbage)
__device__ __forceinline__ void trace_stamp(int row, int& n) {
  if (blockIdx.x == 0 && n < 512) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    g_trace[row][n] = t;
  }
  ++n;
}
#ifdef TEMCO_NOSTAMP
#define TRACE(row, n) ((void)0)
#else
#define TRACE(row, n) trace_stamp(row, n)
#endif
// cycle accounting of CTA 0's MMA issuer: waits by kind, op loads, total
__device__ unsigned long long g_prof[64][16];   // per wide-kernel launch (launch order)
__device__ int g_prof_n;
#define PROF_T0() (_pt0 = clock64())
#define PROF_ADD(var) (var += clock64() - _pt0)
#else
#define TRACE(row, n) ((void)0)
#define PROF_T0() ((void)0)
#define PROF_ADD(var) ((void)0)
#endif

// 32 consecutive fp32 values (16-byte aligned) -> registers
__device__ __forceinline__ void load_bias32(const float* src, float (&b)[32]) {
  const float4* s4 = reinterpret_cast<const float4*>(src);
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const float4 v = __ldg(s4 + i);
    b[4 * i] = v.x;
    b[4 * i + 1] = v.y;
    b[4 * i + 2] = v.z;
    b[4 * i + 3] = v.w;
  }
}

constexpr int kEpiWarps = 8;
constexpr int kProdWarp = 8, kMmaWarp = 9;
constexpr int kThreads = 32 * 10;

// Units of one tile: pooled chunks c < npc contribute ntg tap-group units each,
// every other chunk one unit.  Units are processed in pairs (TMEM buffers 0, 1);
// all roles walk the same order: for pair: for level: for unit in pair.
struct Unit {
  int c, tg, nt;      // chunk, tap group, taps in the unit (1 for plain chunks)
  bool pooled, last;  // pooled-member chunk; last unit of its chunk
};

__device__ __forceinline__ int units_per_tile(const TcChainDesc& d) { return d.npc * d.ntg + d.nchunks - d.npc; }

__device__ __forceinline__ Unit unit_at(const TcChainDesc& d, int u) {
  Unit x;
  if (u < d.npc * d.ntg) {
    x.c = u / d.ntg;
    x.tg = u % d.ntg;
    x.nt = min(d.tpu, d.mtaps - x.tg * d.tpu);
    x.pooled = true;
    x.last = x.tg == d.ntg - 1;
  } else {
    x.c = d.npc + (u - d.npc * d.ntg);
    x.tg = 0;
    x.nt = 1;
    x.pooled = false;
    x.last = true;
  }
  return x;
}

struct TileGeo {
  int m0, n0, h0, w0;
};

__device__ __forceinline__ TileGeo tile_geo(const TcChainDesc& d, int tile) {
  TileGeo g{tile * d.rows_per_tile, 0, 0, 0};
  if (d.spatial) {
    const int per_img = d.nhb * d.nwb;
    const int nb = tile / per_img, rem = tile % per_img;
    g.n0 = nb * d.tn;
    g.h0 = (rem / d.nwb) * d.th;
    g.w0 = (rem % d.nwb) * d.tw;
  }
  return g;
}

// pooled-member activation: ReLU when a != 0; SILU instantiation: a == 2 -> SiLU
template <bool SILU>
__device__ __forceinline__ float act_m(float x, int a) {
  if constexpr (SILU) return a == 2 ? silu_fast(x) : (a ? fmaxf(x, 0.f) : x);
  else return a ? fmaxf(x, 0.f) : x;
}

template <bool SILU>
__global__ void __launch_bounds__(kThreads, 1) tc_wide_kernel(const __grid_constant__ TcChainDesc d, RunPtrs p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  const int S = d.stages;
  const int kSlotA = d.slot_a;
  const int slot = kSlotA + d.slot_b;
  const int Cc = d.Cc;
  const int pbytes = 128 * Cc * 2;
  uint8_t* wres = smem;                    // resident weights (d.resident), else empty
  uint8_t* ring = smem + d.wres_bytes;
  uint8_t* pbuf = ring + S * slot;
  uint8_t* ones = pbuf + 2 * pbytes;
  uint8_t* zeros = ones + 4096;            // zero B tile (zero-init MMA of a region no term reaches)
  uint64_t* bars = reinterpret_cast<uint64_t*>(zeros + 4096);
  uint64_t* full = bars;
  uint64_t* empty = bars + S;
  uint64_t* acc_full = bars + 2 * S;
  uint64_t* acc_empty = acc_full + 2;
  uint64_t* p_full = acc_empty + 2;
  uint64_t* p_empty = p_full + 2;
  uint64_t* out_full = p_empty + 2;
  uint64_t* out_empty = out_full + 1;
  uint64_t* wbar = out_empty + 1;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(wbar + 1);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  // constant A operand of the bias MMA: K columns 0 and 1 = 1.0 (bf16), one SW32 atom
  for (int i = threadIdx.x; i < 128 * 2; i += blockDim.x) {
    const int row = i / 2, ch = i % 2;
    uint4 v = make_uint4(0, 0, 0, 0);
    if (ch == swz_chunk(row, 0, 16)) v.x = 0x3F803F80u;   // logical chunk 0 of this row
    reinterpret_cast<uint4*>(ones)[i] = v;
  }
  for (int i = threadIdx.x; i < 4096 / 16; i += blockDim.x) reinterpret_cast<uint4*>(zeros)[i] = make_uint4(0, 0, 0, 0);
  fence_proxy_async();
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&acc_full[b], 1);
      mbar_init(&acc_empty[b], kEpiWarps);
      mbar_init(&p_full[b], kEpiWarps);
      mbar_init(&p_empty[b], 1);
    }
    mbar_init(out_full, 1);
    mbar_init(out_empty, kEpiWarps);
    mbar_init(wbar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  // per-tile programs -> SMEM
  const TcProdOp* prod = d.prod;
  const TcMmaOpD* mprog = d.mma;
  if (d.prog_smem) {
    uint8_t* ps = reinterpret_cast<uint8_t*>(bars) + 2048 + (d.npc ? 32768 : 0);
    const int n16 = (d.n_prod * (int)sizeof(TcProdOp) + d.n_mma * (int)sizeof(TcMmaOpD)) / 16;
    const uint4* src = reinterpret_cast<const uint4*>(d.prod);
    for (int i = threadIdx.x; i < n16; i += blockDim.x) reinterpret_cast<uint4*>(ps)[i] = src[i];
    prod = reinterpret_cast<const TcProdOp*>(ps);
    mprog = reinterpret_cast<const TcMmaOpD*>(ps + d.n_prod * sizeof(TcProdOp));
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
  pdl_wait();
  pdl_trigger_early();
  const int U = units_per_tile(d);

  const int rows_atom = d.spatial ? d.tw * d.th * d.tn : 128;   // rows of one A box
  if (warp == kProdWarp) {
    // ------------------------------------------------------------ TMA producer
    {   // whole warp; one elected lane issues (the resident preload runs in lane 0)
      int stage = 0;
      uint32_t phase = 0;
      [[maybe_unused]] int n0 = 0, n1 = 0;
      const char* dbase = reinterpret_cast<const char*>(&d);
      if (d.resident && lane == 0) {
        // every B box once: term atoms, level / member biases, F atoms
        mbar_expect_tx(wbar, d.wres_bytes);
        const int nall = d.npc ? d.mt1 : d.n_terms;
        for (int j = 0; j < nall; ++j) {
          const TcTerm& t = d.term[j];
          const int ka_n = t.Rp / t.aw, bb = Cc * t.aw * 2;
          for (int c = 0; c < t.nhit; ++c)
            for (int ka = 0; ka < ka_n; ++ka)
              tma_load_2d(wres + t.wres + (c * ka_n + ka) * bb, t.wmap, wbar, ka * t.aw, (t.cfirst + c) * Cc);
        }
        if (!d.gap)
          for (int a = 0; a < d.Cpad / 64; ++a) tma_load_2d(wres + d.fres + a * d.Np * 128, d.fmap, wbar, a * 64, 0);
      }
      __syncwarp();
      const int np = d.n_prod;
      for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x) {
        const TileGeo gg = tile_geo(d, tile);
        for (int i = 0; i < np; ++i) {
          const TcProdOp o = prod[i];
#ifdef TEMCO_TRACE
          if (g_dbg & 1) {   // TMA-only experiment: the producer recycles its own stages
            if (n0 >= S) mbar_wait(&full[stage], phase ^ 1);
          } else
#endif
          mbar_wait(&empty[stage], phase ^ 1);
          TRACE(0, n0);
          mbar_expect_tx_w(&full[stage], o.bytes);
          uint8_t* sa = ring + stage * slot;
          for (int a = 0; a < (int)o.n2; ++a) {   // one or two K atoms per stage
            const int aoffb = a * rows_atom * o.aw * 2, boffb = a * o.bstep64 * 64, ka = a * o.aw;
            if (o.kind & PK_A4D)        // (tap-shifted) strided box of the term's input
              tma_load_4d_w(sa + aoffb, dbase + o.amap * 64, &full[stage], o.ac + ka, gg.w0 * o.ts + o.dx,
                            gg.h0 * o.ts + o.dy, gg.n0);
            else if (o.kind & PK_A2D)
              tma_load_2d_w(sa + aoffb, dbase + o.amap * 64, &full[stage], o.ac + ka, gg.m0);
            if (o.kind & PK_B) tma_load_2d_w(sa + kSlotA + boffb, dbase + o.bmap * 64, &full[stage], o.bx + ka, o.by);
          }
          TRACE(1, n1);
          if (++stage == S) stage = 0, phase ^= 1;
        }
      }
#ifdef TEMCO_TRACE
      if ((g_dbg & 1) && lane == 0)
        for (int k = 0; k < S && k < n0; ++k) {
          const int i = n0 - 1 - k;
          mbar_wait(&full[i % S], (i / S) & 1);
        }
#endif
    }
  } else if (warp == kMmaWarp) {
#ifdef TEMCO_TRACE
    if (g_dbg & 1) goto done;
#endif
    // ------------------------------------------------------------ MMA issuer
    {   // whole warp (uniform control flow); elect.sync picks the issuing lane
      int stage = 0;
      uint32_t phase = 0;
      uint32_t acc_par = 0, p_par = 0, tile_iter = 0;   // phase parity bits per buffer (registers only)
      [[maybe_unused]] int n2 = 0, n3 = 0, n8 = 0, n9 = 0, n10 = 0, n11 = 0;
      if (d.resident) mbar_wait(wbar, 0);
      const int nm = d.n_mma;
#ifdef TEMCO_TRACE
      long long pc_acc = 0, pc_p = 0, pc_out = 0, pc_full = 0, pc_issue = 0, pc_n = 0, pc_dec = 0, pc_com = 0;
      const long long pc_start = clock64();
#endif
      const uint64_t base16 = smem_u32(smem) >> 4;
      auto exec = [&](const TcMmaOpD o, int gu, uint32_t tile_iter) {   // by value: one LDS.128 pair, then registers
#ifdef TEMCO_TRACE
          long long _pt0 = 0;
#endif
          const uint32_t f = o.flags;
          const int bs = (gu + o.unit) & 1;
          if (f & MF_ACC_WAIT) {
            PROF_T0();
            mbar_wait(&acc_empty[bs], ((acc_par >> bs) & 1u) ^ 1u);
            PROF_ADD(pc_acc);
            TRACE(8, n8);
            tc_fence_after();
          }
          if (f & MF_P_WAIT) {
            TRACE(9, n9);
            PROF_T0();
            mbar_wait(&p_full[o.unit], (p_par >> o.unit) & 1u);
            PROF_ADD(pc_p);
            TRACE(10, n10);
            tc_fence_after();
          }
          if (f & MF_OUT_WAIT) {
            PROF_T0();
            mbar_wait(out_empty, (tile_iter & 1) ^ 1);
            PROF_ADD(pc_out);
            tc_fence_after();
          }
          if (f & MF_SW) {
            PROF_T0();
            mbar_wait(&full[stage], phase);
            PROF_ADD(pc_full);
            TRACE(2, n2);
            tc_fence_after();
          }
          PROF_T0();
          const uint64_t st16 = (uint64_t)((stage * slot) >> 4);
          const uint64_t ad = o.adesc + base16 + ((f & MF_SA) ? st16 : 0);
          const uint64_t bd = o.bdesc + base16 + ((f & MF_SB) ? st16 : 0);
          const uint32_t dt = tbase + (o.tmem & 0xFFFFu) + ((f & MF_F) ? 0u : (uint32_t)(bs * d.ubuf));
          const uint32_t nk1 = (o.tmem >> 24) ? (o.tmem >> 24) : 8u;   // steps in the stage's first atom
          const uint32_t acc0 = (f & MF_ZERO) ? 0u : 1u;
          PROF_ADD(pc_dec);
          {
          PROF_T0();
          // K=16 steps of the op (nk <= 4), unrolled: descriptors advance by 32 bytes (>> 4 = 2)
          const uint32_t idesc = o.idesc, nk = o.nk;
          mma_bf16_w(dt, ad, bd, idesc, acc0);
#pragma unroll
          for (uint32_t k = 1; k < 8; ++k)
            if (k < nk) {
              const bool second = k >= nk1;   // second atom of a two-atom stage
              const uint32_t kk = second ? k - nk1 : k;
              mma_bf16_w(dt, ad + (second ? o.a2 : 0) + 2 * kk, bd + (second ? o.b2 : 0) + 2 * kk, idesc, 1u);
            }
          PROF_ADD(pc_issue);
#ifdef TEMCO_TRACE
          pc_n += o.nk;
#endif
          }
          PROF_T0();
          if (f & MF_SD) {
            mma_commit_w(&empty[stage]);
            if (++stage == S) stage = 0, phase ^= 1;
          }
          if (f & MF_ACC_COMMIT) {
            mma_commit_w(&acc_full[bs]);
            TRACE(3, n3);
            acc_par ^= 1u << bs;
          }
          if (f & MF_P_COMMIT) {
            mma_commit_w(&p_empty[o.unit]);
            p_par ^= 1u << o.unit;
          }
          if (f & MF_OUT_COMMIT) {
            mma_commit_w(out_full);
            TRACE(11, n11);
          }
          PROF_ADD(pc_com);
      };
      if (d.mma_head > 0) {
        // software pipeline over tiles: the unit ops of tile t+1 go ahead of the
        // fconv ops of tile t (which wait for the epilogue's P tile of t)
        const int nh = d.mma_head;
        int t = blockIdx.x, gu = 0;
        for (int i = 0; i < nh && t < d.ntiles; ++i) exec(mprog[i], gu, tile_iter);
        for (; t < d.ntiles; t += gridDim.x) {
          if (t + (int)gridDim.x < d.ntiles)
            for (int i = 0; i < nh; ++i) exec(mprog[i], gu + d.units, tile_iter + 1);
          for (int i = nh; i < nm; ++i) exec(mprog[i], gu, tile_iter);
          gu += d.units;
          ++tile_iter;
        }
      } else {
        int gu = 0;   // units issued so far (TMEM buffer parity)
        for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x) {
          for (int i = 0; i < nm; ++i) exec(mprog[i], gu, tile_iter);
          gu += d.units;
          ++tile_iter;
        }
      }
#ifdef TEMCO_TRACE
      if (blockIdx.x == 0 && lane == 0) {
        const int li = atomicAdd(&g_prof_n, 1) & 63;
        g_prof[li][0] = clock64() - pc_start;
        g_prof[li][1] = pc_acc;
        g_prof[li][2] = pc_p;
        g_prof[li][3] = pc_out;
        g_prof[li][4] = pc_full;
        g_prof[li][5] = pc_issue;
        g_prof[li][6] = pc_n;
        g_prof[li][7] = pc_dec;
        g_prof[li][8] = pc_com;
        g_prof[li][9] = d.ntiles;
        g_prof[li][10] = d.units;
        g_prof[li][11] = d.stages;
      }
#endif
    }
  } else if (warp < kEpiWarps) {
#ifdef TEMCO_TRACE
    if (g_dbg & 1) goto done;
#endif
    // ------------------------------------------------------------ epilogue (8 warps)
    // warp w: TMEM lane quarter q = w % 4 (pixel rows 32q..32q+31), column half h = w / 4
    const int q = warp & 3, h = warp >> 2;
    const int row = q * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    const int half = Cc / 2;                          // columns per warp (32 or 64)
    const int c_lo = h * half;
    uint32_t acc_par = 0, p_par = 0, tile_iter = 0;   // phase parity bits per buffer (registers only)
    [[maybe_unused]] int n4 = 0, n5 = 0, n6 = 0, n7 = 0;
    const bool tr = threadIdx.x == 0;
    (void)tr;
    __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.arena + d.y.off);
    float* runbuf = reinterpret_cast<float*>(bars + 64);   // pooled member running max / sum (32 KB)
    int gu = 0;   // units consumed so far (TMEM buffer parity)
    for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x) {
      int64_t m = (int64_t)tile * d.rows_per_tile + row;
      bool mvalid = m < d.npix;
      int ho = 0, wo = 0;
      if (d.spatial) {
        // spatial tile: row -> (image, output row, output column)
        const TileGeo gg = tile_geo(d, tile);
        const int ni = row / (d.tw * d.th), hi = (row / d.tw) % d.th, wi = row % d.tw;
        const int n = gg.n0 + ni;
        ho = gg.h0 + hi;
        wo = gg.w0 + wi;
        mvalid = row < d.mused && n < d.nimg && ho < d.Ho && wo < d.Wo;
        m = ((int64_t)n * d.Ho + ho) * d.Wo + wo;
      }
      for (int u0 = 0; u0 < U; gu += min(2, U - u0), u0 += 2) {
        const int nb = min(2, U - u0);
        for (int l = 0; l < d.n_levels; ++l) {
          const bool last = l == d.n_levels - 1;
          const int relu = d.relu[l];   // 0 none, 1 ReLU, 2 SiLU (SILU instantiation only)
          for (int bi = 0; bi < nb; ++bi) {
            const Unit un = unit_at(d, u0 + bi);
            const int bs = (gu + bi) & 1;
            const uint32_t abit = 1u << bs;
            mbar_wait(&acc_full[bs], (acc_par & abit) ? 1u : 0u);
            if (tr) TRACE(4, n4);
            acc_par ^= abit;
            tc_fence_after();
            const int pb = un.c & 1;
            const bool writes_p = last && !d.gap && un.last;
            if (writes_p) {
              const uint32_t pbit = 1u << pb;
              mbar_wait(&p_empty[pb], ((p_par & pbit) ? 1u : 0u) ^ 1u);
              p_par ^= pbit;
            }
            const uint32_t ta = tbase + lane_off + bs * d.ubuf + c_lo;
            uint8_t* P = pbuf + pb * pbytes;
            // level / member bias (fp32, added here rather than through the tensor core)
            const float* bsrc = p.params + (un.pooled ? d.mbias : d.lbias[l]) + un.c * Cc + c_lo;
#ifdef TEMCO_TRACE
            if (g_dbg & 2) {   // experiment: epilogue does no TMEM / SMEM work
            } else
#endif
            if (un.pooled) {
              // pooled member: fold the unit's taps into the running max / sum (half == 32);
              // registers within the unit, a conflict-free SMEM slab across units
              // (element i of thread t at run[i * 256 + t])
              float* run = runbuf + threadIdx.x;
              float cur[32];
              const float4* b4 = reinterpret_cast<const float4*>(bsrc);
              const bool fresh = un.tg == 0;
#pragma unroll
              for (int i = 0; i < 32; ++i) cur[i] = fresh ? (d.mpool == 1 ? -INFINITY : 0.f) : run[i * 256];
              for (int r = 0; r < un.nt; ++r) {
                const int tap = un.tg * d.tpu + r;
                const int hi = ho * d.ms - d.mp + tap / d.mk, wi = wo * d.ms - d.mp + tap % d.mk;
                const bool valid = hi >= 0 && hi < d.mHin && wi >= 0 && wi < d.mWin;
                uint32_t v[32];
                tmem_ld32(ta + r * Cc, v);
                tmem_wait_ld();
#pragma unroll
                for (int i4 = 0; i4 < 8; ++i4) {
                  const float4 bb = __ldg(b4 + i4);
                  const float bq[4] = {bb.x, bb.y, bb.z, bb.w};
#pragma unroll
                  for (int k = 0; k < 4; ++k) {
                    const int i = 4 * i4 + k;
                    float x = __uint_as_float(v[i]) + bq[k];
                    x = act_m<SILU>(x, d.mrelu);
                    if (d.mpool == 1)
                      cur[i] = valid ? fmaxf(cur[i], x) : cur[i];
                    else
                      cur[i] += x;
                  }
                }
              }
              if (!un.last) {
#pragma unroll
                for (int i = 0; i < 32; ++i) run[i * 256] = cur[i];
              } else {
                // pooled value, + post-pool shift (BN after the pool), level activation
                const float sc = d.mpool == 2 ? 1.f / (float)d.mtaps : 1.f;
                const float4* pv4 = reinterpret_cast<const float4*>(p.params + (d.post >= 0 ? d.post : d.mbias) + un.c * Cc + c_lo);
                const float pscale = d.post >= 0 ? 1.f : 0.f;
                const float* psc = p.params + (d.postsc >= 0 ? d.postsc : 0) + un.c * Cc + c_lo;
                const int ch0 = c_lo / 8;
#pragma unroll
                for (int qq = 0; qq < 4; ++qq) {
                  float f[8];
                  const float4 pa = __ldg(pv4 + 2 * qq), pb2 = __ldg(pv4 + 2 * qq + 1);
                  const float pq[8] = {pa.x, pa.y, pa.z, pa.w, pb2.x, pb2.y, pb2.z, pb2.w};
#pragma unroll
                  for (int i = 0; i < 8; ++i) {
                    const float ms = d.postsc >= 0 ? __ldg(psc + 8 * qq + i) : 1.f;
                    const float x = cur[8 * qq + i] * sc * ms + pscale * pq[i];
                    f[i] = act_w<SILU>(x, relu);
                  }
                  uint4 pk;
                  pk.x = pack_bf16(f[0], f[1]);
                  pk.y = pack_bf16(f[2], f[3]);
                  pk.z = pack_bf16(f[4], f[5]);
                  pk.w = pack_bf16(f[6], f[7]);
                  *reinterpret_cast<uint4*>(P + row * 128 + (((ch0 + qq) ^ (row & 7)) * 16)) = pk;
                }
              }
            } else if (!last) {
              // t_l = relu(acc + b_l) back into TMEM for the next level's MMAs
              for (int g = 0; g < half / 32; ++g) {
                uint32_t a[32];
                float bv[32];
                load_bias32(bsrc + g * 32, bv);
                tmem_ld32(ta + g * 32, a);
                tmem_wait_ld();
#pragma unroll
                for (int i = 0; i < 32; ++i) {
                  const float x = __uint_as_float(a[i]) + bv[i];
                  a[i] = __float_as_uint(act_w<SILU>(x, relu));
                }
                tmem_st32(ta + g * 32, a);
              }
              tmem_wait_st();
            } else if (d.gap) {
              // GAP root: per-image column means; tiles hold whole images so the
              // summation order is fixed (deterministic, batch-invariant)
              float* red = reinterpret_cast<float*>(pbuf + h * pbytes);
              for (int g = 0; g < half / 32; ++g) {
                uint32_t v[32];
                float bv[32];
                load_bias32(bsrc + g * 32, bv);
                tmem_ld32(ta + g * 32, v);
                tmem_wait_ld();
#pragma unroll
                for (int i = 0; i < 32; ++i) {
                  const float x0 = __uint_as_float(v[i]) + bv[i];
                  const float x = act_w<SILU>(x0, relu);
                  red[row * 32 + ((i + row) & 31)] = x;
                }
                asm volatile("bar.sync %0, 128;" ::"r"(1 + h) : "memory");
                for (int idx = row; idx < d.ipt * 32; idx += 128) {
                  const int ii = idx / 32, col = idx % 32;
                  const int n = tile * d.ipt + ii;
                  float acc = 0.f;
                  for (int r = ii * d.hw; r < (ii + 1) * d.hw; ++r) acc += red[r * 32 + ((col + r) & 31)];
                  const int cg = un.c * Cc + c_lo + g * 32 + col;
                  if (n < d.nimg && cg < d.C) y[(int64_t)n * d.C + cg] = __float2bfloat16_rn(acc / (float)d.hw);
                }
                asm volatile("bar.sync %0, 128;" ::"r"(1 + h) : "memory");
              }
            } else {
              // last level: P = bf16 relu(acc + b) -> SMEM (SW128 K-major atoms of 64 columns)
              for (int g = 0; g < half / 32; ++g) {
                uint32_t v[32];
                float bv[32];
                load_bias32(bsrc + g * 32, bv);
                tmem_ld32(ta + g * 32, v);
                tmem_wait_ld();
                const int col = c_lo + g * 32;
                uint8_t* atom = P + (col / 64) * 16384 + row * 128;
                const int ch0 = (col % 64) / 8;
#pragma unroll
                for (int qq = 0; qq < 4; ++qq) {
                  float f[8];
#pragma unroll
                  for (int i = 0; i < 8; ++i) {
                    const float x = __uint_as_float(v[8 * qq + i]) + bv[8 * qq + i];
                    f[i] = act_w<SILU>(x, relu);
                  }
                  uint4 pk;
                  pk.x = pack_bf16(f[0], f[1]);
                  pk.y = pack_bf16(f[2], f[3]);
                  pk.z = pack_bf16(f[4], f[5]);
                  pk.w = pack_bf16(f[6], f[7]);
                  *reinterpret_cast<uint4*>(atom + (((ch0 + qq) ^ (row & 7)) * 16)) = pk;
                }
              }
            }
            tc_fence_before();
            if (tr) TRACE(5, n5);
            warp_arrive(&acc_empty[bs]);
            if (writes_p) {
              fence_proxy_async();
              warp_arrive(&p_full[pb]);
            }
          }
        }
      }
      if (d.gap) continue;
      // output epilogue: column groups of 8 split between the two warp halves
      if (tr) TRACE(6, n6);
      mbar_wait(out_full, tile_iter & 1);
      if (tr) TRACE(7, n7);
      ++tile_iter;
      tc_fence_after();
      const int ng = d.Np / 8, gh = (ng + 1) / 2;
#ifdef TEMCO_TRACE
      const int gend = (g_dbg & 2) ? 0 : min(ng, (h + 1) * gh);
#else
      const int gend = min(ng, (h + 1) * gh);
#endif
      for (int g = h * gh; g < gend; ++g) {
        uint32_t v[8];
        tmem_ld8(tbase + lane_off + 2 * d.ubuf + g * 8, v);
        tmem_wait_ld();
        if (mvalid && g * 8 < d.Nout) {
          uint4 pk;
          pk.x = pack_bf16(__uint_as_float(v[0]), __uint_as_float(v[1]));
          pk.y = pack_bf16(__uint_as_float(v[2]), __uint_as_float(v[3]));
          pk.z = pack_bf16(__uint_as_float(v[4]), __uint_as_float(v[5]));
          pk.w = pack_bf16(__uint_as_float(v[6]), __uint_as_float(v[7]));
          *reinterpret_cast<uint4*>(y + m * d.Nout + g * 8) = pk;
        }
      }
      tc_fence_before();
      warp_arrive(out_empty);
    }
  }
#ifdef TEMCO_TRACE
done:
#endif
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
    cudaFuncSetAttribute(tc_wide_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    cudaFuncSetAttribute(tc_wide_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    configured = true;
  }
  int grid = std::min(d.ntiles, sms > 0 ? sms : 148);
  static const int grid_cap = getenv("TEMCO_TC_GRID") ? atoi(getenv("TEMCO_TC_GRID")) : 0;   // experiments
  if (grid_cap > 0) grid = std::min(grid, grid_cap);
  // >= 114 KB of shared memory keeps one CTA per SM (each may own all 512 TMEM columns)
  const bool silu = d.mrelu == 2 || std::any_of(d.relu, d.relu + d.n_levels, [](int32_t a) { return a == 2; });
  launch_pdl(silu ? tc_wide_kernel<true> : tc_wide_kernel<false>, dim3(grid), dim3(kThreads),
             std::max(d.smem_bytes, 116 * 1024), s, d, p);
}

}  // namespace wide
}  // namespace temco

#ifdef TEMCO_TRACE
// experiment builds: CTA 0 MMA-issuer cycle accounting of each wide-kernel launch since the last call
extern "C" int temco_debug_wide_prof(unsigned long long* out) {
  int n = 0;
  cudaMemcpyFromSymbol(&n, temco::wide::g_prof_n, sizeof(int));
  cudaMemcpyFromSymbol(out, temco::wide::g_prof, sizeof(unsigned long long) * 64 * 16);
  const int z = 0;
  cudaMemcpyToSymbol(temco::wide::g_prof_n, &z, sizeof(int));
  return n;
}
extern "C" void temco_debug_wide_dbg(int v) { cudaMemcpyToSymbol(temco::wide::g_dbg, &v, sizeof(int)); }
#endif
