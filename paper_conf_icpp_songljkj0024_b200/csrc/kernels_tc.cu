// tcgen05 fused restore-chain -> BN -> add/concat -> ReLU -> [pool] -> reduce kernel (sm_100a).
//
// One fused group computes, per output tile of 128 pixels,
//     t_l = act_l( sum_{j in l} r_j Lhat_j^T + b_l + t_{l-1} ),  out = t_D F^T
// with the C-wide t never leaving the SM.  The restored width is cut into units
// of 64 channels; a unit's levels are evaluated back to back:
//   GEMM1  r_j atoms [rows x aw] (2D TMA of 128 consecutive pixels, or 4D TMA of
//          a tap-shifted, strided spatial box) x Lhat_j atoms [64 x aw] (TMA,
//          SMEM-resident when they fit) -> tcgen05.mma (M=128, N=64) into a
//          fresh TMEM accumulator slot per (unit, level); slots form a ring, so
//          the MMA issuer runs ahead of the epilogue by several unit-levels.
//   level epilogue: TMEM -> registers, + b_l + t_{l-1} (t lives in registers:
//          no tcgen05.st round trip), ReLU; the slot is released as soon as it
//          has been read.  After the last level the bf16 tile P = t_D goes to
//          SMEM in the SW128 K-major layout.  Pooled-member units keep one TMEM
//          region per tap and fold max / sum in registers; GAP roots reduce per
//          image.
//   GEMM2  tcgen05.mma (A = P, B = F atom) accumulates out over the units in
//          a TMEM output buffer; the output epilogue stores bf16 rows.
// Warp roles (640 threads, persistent over tiles): warps 0-15 epilogue in two
// teams of 8 that take alternate tiles (one team's TMEM-load latency hides
// behind the other's arithmetic); warp 16 TMA producer (A / B ring), 17 GEMM1
// issuer, 18 GEMM2 issuer, 19 F-ring producer (and TMEM allocation).
#include <cuda.h>
#include <cuda_bf16.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cmath>
#include <set>

#include "tmap.h"
#include "chain_lower.h"
#include "chain_parse.h"
#include "tc.h"
#include "tc_ptx.cuh"

namespace temco {

// ===========================================================================
// host: lowering
// ===========================================================================
namespace {
using namespace chainp;
using chainl::push_bf16;
using chainl::push_f32;
using chainl::to_bf16;




struct HUnit {
  int c, tg, nt;
  bool pooled, last;
};

HUnit unit_of(const TcChainDesc& d, int u) {
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
}

// Per-tile producer / MMA programs.  Producer: every distinct A atom of the
// tile (term x tap x K atom) once into the tile's A buffer, then (B streamed)
// one ring stage per MMA op.  MMA order: for each unit: for each of its levels
// (pooled units: one): [terms x taps x K atoms] into one accumulator slot.
void build_programs(TcChainDesc& d, std::vector<uint16_t>& tcw) {
  std::vector<TcProdOp> P, PB;
  std::vector<TcMmaOp> M;
  const int Cc = d.Cc;
  const int U = d.npc * d.ntg + d.nchunks - d.npc;
  d.units = U;
  const bool res = d.resident != 0;
  const int rows_a = d.spatial ? d.tw * d.th * d.tn : 128;
  auto moff = [&](const unsigned char* m) {
    return (uint16_t)((reinterpret_cast<const char*>(m) - reinterpret_cast<const char*>(&d)) / 64);
  };
  std::map<std::tuple<int, int, int>, uint32_t> atom;   // (term, tap, K atom) -> offset in the A buffer
  uint32_t aoff = 0;
  int atx = 0;
  auto atom_of = [&](int j, int tap, int ka, int kk, int pad) {
    const auto key = std::make_tuple(j, tap, ka);
    auto it = atom.find(key);
    if (it != atom.end()) return it->second;
    const TcTerm& t = d.term[j];
    TcProdOp o{};
    o.kind = d.spatial ? PK_A4D : PK_A2D;
    o.ts = (uint8_t)t.ts;
    o.amap = moff(d.spatial ? t.tmap4 : t.tmap);
    o.ac = (int16_t)(ka * t.aw);
    o.dx = (int16_t)(tap % kk - pad);
    o.dy = (int16_t)(tap / kk - pad);
    o.bytes = (uint16_t)(rows_a * t.aw * 2);
    o.dst = aoff;
    P.push_back(o);
    atx += rows_a * t.aw * 2;
    const uint32_t off = aoff;
    aoff += (uint32_t)((rows_a * t.aw * 2 + 1023) / 1024 * 1024);
    atom[key] = off;
    return off;
  };
  int spt = 0;
  for (int u = 0; u < U; ++u) {
    const HUnit un = unit_of(d, u);
    const int nl = un.pooled ? 1 : d.n_levels;
    for (int l = 0; l < nl; ++l) {
      ++spt;
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
            for (int ka = 0; ka < katoms; ++ka) {
              TcMmaOp m{};
              m.aoff = atom_of(j, tap, ka, kk, pad);
              m.flags = MF_AT | (res ? MF_BRES : MF_SW | MF_SB | MF_SD);
              if (!res) {
                TcProdOp o{};
                o.kind = PK_B;
                o.bmap = moff(t.wmap);
                o.bx = (int16_t)(ka * t.aw);
                o.by = (int16_t)(un.c * Cc);
                o.bytes = (uint16_t)(Cc * t.aw * 2);
                PB.push_back(o);
              }
              if (!region_done[r]) m.flags |= MF_ZERO;
              region_done[r] = 1;
              m.nk = (uint8_t)std::min(t.aw / 16, (t.R - ka * t.aw + 15) / 16);
              m.la = (uint8_t)t.aw;
              m.lb = (uint8_t)t.aw;
              m.tcol = (uint16_t)(r * Cc);
              if (res) m.boff = (uint32_t)(t.wres + ((un.c - t.cfirst) * katoms + ka) * Cc * t.aw * 2);
              M.push_back(m);
            }
          }
        }
      for (int r = 0; r < un.nt; ++r)
        if (!region_done[r]) {   // zero-init: ones tile x zero tile
          TcMmaOp m{};
          m.flags = MF_ONES | MF_BZERO | MF_ZERO;
          m.nk = 1;
          m.la = 16;
          m.lb = 16;
          m.tcol = (uint16_t)(r * Cc);
          M.push_back(m);
        }
      M[m_first].flags |= MF_ACC_WAIT;
      M.back().flags |= MF_ACC_COMMIT;
    }
  }
  d.n_aload = (int32_t)P.size();
  d.a_tx = atx;
  for (const TcProdOp& o : PB) P.push_back(o);
  d.spt = spt;
  d.n_prod = (int32_t)P.size();
  d.n_mma = (int32_t)M.size();
  while (tcw.size() % 512) tcw.push_back(0);
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
    const uint32_t aoff = (m.flags & MF_ONES) ? (uint32_t)d.off_ones : (uint32_t)d.off_abuf + m.aoff;
    const uint32_t boff = (m.flags & MF_BZERO) ? (uint32_t)d.off_zeros
                          : (m.flags & MF_BRES) ? m.boff
                                                : (uint32_t)d.off_ring;
    o.adesc = dtmpl(aoff, m.la);
    o.bdesc = dtmpl(boff, m.lb);
    o.idesc = idesc(128, Cc);
    o.tmem = m.tcol;
    o.flags = m.flags;
    o.nk = m.nk;
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
  // store root: the group's value itself is the output (e.g. VGG's last pooled
  // block feeding the classifier), written as bf16 NHWC without a fconv
  const bool store = !gap && root.role != ROLE_FCONV;
  if (!store && !gap && root.b) return false;    // fconv factors carry no bias (O1)
  const int tsrc = store ? s.out : ir.oin[s.out][0];
  const Node& tn = ir.nodes[tsrc];
  const int C = tn.C, Nout = (gap || store) ? 16 : root.C;
  if (Nout % 8 || Nout > 256) return false;
  if (gap && tn.H * tn.W > 128) return false;
  if (store && C % kTcCc) return false;
  ChainParser P{ir, std::set<int>(s.members.begin(), s.members.end()), C, {}, tn.H, tn.W};
  P.allow_silu = true;   // d.relu[l]: 1 ReLU, 2 SiLU
  if (!store) P.members.erase(s.out);
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
  if (pm && (pm->c0 != 0 || pm->C % kTcCc)) return false;
  if (pm && gap) return false;                       // GAP over a max-pooled member: generic path
  const bool nogemm2 = gap || store;
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
  d.Cc = kTcCc;
  if (!chainl::tile_geometry(d, ir, tn, Nout, gap, mixed, yl, (int)levels.size())) return false;
  int64_t flops = 0, bytes = 0;
  int j = 0;
  auto add_term = [&](const PTerm& t) -> bool { return chainl::add_term(d, d.term[j++], ir, loc, tcw, t, flops, bytes); };
  for (int l = 0; l < d.n_levels; ++l) {
    const PLevel& L = levels[l];
    d.relu[l] = L.relu ? 1 : L.silu ? 2 : 0;
    // pooled-member channels take no level bias before the pool: their level
    // bias (the post-BN shift) is added after pooling, in the epilogue
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
    d.mbias = push_f32(params, pm->bias, d.Cpad);
    if (d.tw * d.ms > 256 || d.th * d.ms > 256) return false;
  }
  d.F = 0;
  d.store = store ? 1 : 0;
  if (gap) {
    d.alg_flops = flops + d.npix * C;
    d.alg_bytes = bytes + 2LL * ir.batch * C;
  } else if (store) {
    d.alg_flops = flops;
    d.alg_bytes = bytes + d.npix * 2LL * C;
  } else {
    std::vector<float> f((size_t)d.Np * d.Cpad, 0.f);
    for (int o = 0; o < Nout; ++o)
      for (int c = 0; c < C; ++c) f[(size_t)o * d.Cpad + c] = (*root.w)[(size_t)o * C + c];
    d.F = push_bf16(tcw, f);
    d.alg_flops = flops + d.npix * 2LL * Nout * C;
    d.alg_bytes = bytes + d.npix * 2LL * Nout;
  }
  // TMEM: accumulator slots (ubuf columns: one region per tap of a pooled unit)
  // and one or two output buffers of Np columns
  const int npcols = nogemm2 ? 0 : d.Np;
  d.no = nogemm2 ? 0 : (512 - 2 * npcols >= 4 * d.Cc ? 2 : 1);
  const int avail = 512 - d.no * npcols;
  d.tpu = 1;
  d.ntg = 1;
  if (pm) {
    int t = std::max(1, std::min(d.mtaps, avail / (4 * d.Cc)));
    d.ntg = (d.mtaps + t - 1) / t;
    d.tpu = (d.mtaps + d.ntg - 1) / d.ntg;
  }
  d.ubuf = d.tpu * d.Cc;
  d.ns = std::min(8, avail / d.ubuf) & ~1;     // even: each epilogue team owns half the slots
  if (d.ns < 2) return false;
  d.out_col = d.ns * d.ubuf;
  d.tmem_cols = 512;
  // shared memory: [resident weights][A buffers][B ring][F ring][4 P buffers][ones][zeros][barriers][programs]
  const int rows_a = d.spatial ? d.tw * d.th * d.tn : 128;
  int awmax = 16;
  int64_t abytes = 0;
  const int nall = pm ? d.mt1 : d.n_terms;
  for (int i = 0; i < nall; ++i) {
    const TcTerm& T = d.term[i];
    awmax = std::max(awmax, T.aw);
    const int ntap = i >= d.n_terms ? d.mtaps : T.tk * T.tk;
    abytes += (int64_t)ntap * (T.Rp / T.aw) * ((rows_a * T.aw * 2 + 1023) / 1024 * 1024);
  }
  d.atr = 1;
  d.abytes = (int32_t)abytes;
  d.slot_a = 0;
  const int slot_b_stream = (d.Cc * awmax * 2 + 1023) / 1024 * 1024;
  const int fixed = 1024 /*align*/ + 4 * 16384 /*P*/ + 8192 /*ones, zeros*/ + 1024 /*barriers*/;
  const int64_t budget = 227 * 1024 - fixed;
  int64_t wb = 0;
  for (int i = 0; i < nall; ++i) {
    TcTerm& T = d.term[i];
    T.wres = (int32_t)wb;
    wb += (int64_t)T.nhit * (T.Rp / T.aw) * d.Cc * T.aw * 2;
  }
  const int64_t wf = nogemm2 ? 0 : (int64_t)d.nchunks * d.Np * 128;
  d.fslot = nogemm2 ? 0 : (d.Np * 128 + 1023) / 1024 * 1024;
  // first arrangement that fits: two A buffers before one, resident B before
  // resident F; a streamed B needs >= 4 ring stages
  struct Opt { int nab; bool b, f; };
  const Opt opts[8] = {{2, true, true}, {2, true, false}, {2, false, true}, {2, false, false},
                       {1, true, true}, {1, true, false}, {1, false, true}, {1, false, false}};
  bool found = false;
  for (const Opt& o : opts) {
    if (nogemm2 && o.f) continue;
    const int64_t wres = (o.b ? wb : 0) + (o.f ? wf : 0);
    const int64_t wres_al = (wres + 1023) / 1024 * 1024;
    const int fst = (nogemm2 || o.f) ? 0 : 3;
    const int64_t left = budget - wres_al - o.nab * abytes - (int64_t)fst * d.fslot;
    if (left < (o.b ? 0 : 4LL * slot_b_stream)) continue;
    d.nabuf = o.nab;
    d.resident = o.b ? 1 : 0;
    d.fres = o.f ? 1 : 0;
    d.wres_bytes = (int32_t)wres_al;
    d.fbase = (int32_t)(o.b ? wb : 0);
    d.fstages = fst;
    d.slot_b = o.b ? 0 : slot_b_stream;
    d.stages = o.b ? 0 : (int)std::min<int64_t>(24, left / slot_b_stream);
    found = true;
    break;
  }
  // kernel choice (measured on B200): this kernel's 64-channel
  // units issue N=64 MMAs (about half the per-instruction tensor rate of N=128)
  // but keep many small tiles in flight; the wide kernel (N=128, levels
  // accumulated in TMEM) wins for multi-level chains and K >= 128 per unit
  int kmax = 0;
  for (int c = 0; c < d.nchunks; ++c) {
    int k = 0;
    for (int i = 0; i < d.n_terms; ++i) {
      const TcTerm& T = d.term[i];
      if (T.c0 < (c + 1) * d.Cc && T.c0 + T.C > c * d.Cc) k += T.Rp * T.tk * T.tk;
    }
    kmax = std::max(kmax, k);
  }
  bool taps = false;
  for (int i = 0; i < d.n_terms; ++i) taps |= d.term[i].tk > 1;
  const bool prefer_wide = !pm && (d.n_levels >= 2 || (kmax >= 128 && !taps));
  if (getenv("TEMCO_TC_V2") == nullptr && prefer_wide) return false;
  if (!found || getenv("TEMCO_TC_WIDE")) return false;   // -> the wide (TMEM-level) kernel
  d.exp = getenv("TEMCO_TC_EXP") ? atoi(getenv("TEMCO_TC_EXP")) : 0;
  if (getenv("TEMCO_TC_TRACE_OUT") && atoi(getenv("TEMCO_TC_TRACE_OUT")) == s.out) d.exp |= 4;
  d.off_abuf = d.wres_bytes;
  d.off_ring = d.off_abuf + d.nabuf * d.abytes;
  d.off_fring = d.off_ring + d.stages * d.slot_b;
  d.off_p = d.off_fring + d.fstages * d.fslot;
  d.off_ones = d.off_p + 4 * 16384;
  d.off_zeros = d.off_ones + 4096;
  d.off_bars = d.off_zeros + 4096;
  d.off_prog = d.off_bars + 1024;
  d.smem_bytes = 1024 + d.off_prog;
  build_programs(d, tcw);
  // programs live in SMEM when they fit
  const int pbytes_prog = d.n_prod * (int)sizeof(TcProdOp) + d.n_mma * (int)sizeof(TcMmaOpD);
  const int need = (pbytes_prog + 127) / 128 * 128;
  d.prog_smem = 0;
  if (d.smem_bytes + need <= 227 * 1024) {
    d.prog_smem = need;
    d.smem_bytes += need;
  }
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
    if (!d->gap && !d->store && !make(d->fmap, tcw + d->F, (uint64_t)d->Cpad, (uint64_t)d->Np, (uint32_t)d->Np)) {
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

constexpr int kTeamWarps = 8;
constexpr int kEpiWarps = 2 * kTeamWarps;
constexpr int kProdWarp = 16, kMmaWarp = 17, kG2Warp = 18, kFWarp = 19;
constexpr int kThreads = 32 * 20;
constexpr int kTeamArrivals = kTeamWarps;   // one elected arrive per epilogue warp

struct Unit {
  int c, tg, nt;      // chunk, tap group, taps in the unit (1 for plain chunks)
  bool pooled, last;  // pooled-member chunk; last unit of its chunk
};

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

#ifdef TEMCO_TRACE
// experiment builds only: %globaltimer stamps of CTA 0's pipeline events for the
// group lowered with TEMCO_TC_TRACE_OUT=<its output id> (exp bit 4)
constexpr int kTraceRows = 12;
__device__ unsigned long long g_trace[kTraceRows][512];
// per-row event counters live in registers of the stamping thread (tn[row])
#define TRACE(row)                                                              \
  do {                                                                          \
    if ((d.exp & 4) && blockIdx.x == 0 && (threadIdx.x & 31) == 0) {            \
      const int n_ = tn[row]++;                                                 \
      if (n_ < 512) {                                                           \
        unsigned long long t_;                                                  \
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                 \
        g_trace[row][n_] = t_;                                                  \
      }                                                                         \
    }                                                                           \
  } while (0)
#else
#define TRACE(row) ((void)0)
#endif

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

// ring position: stage / parity advance
struct Ring {
  int s;
  uint32_t ph;
  __device__ __forceinline__ void next(int n) {
    if (++s == n) s = 0, ph ^= 1u;
  }
};

// pooled-member activation: ReLU when a != 0; SILU instantiation: a == 2 -> SiLU
template <bool SILU>
__device__ __forceinline__ float act_m(float x, int a) {
  if constexpr (SILU) return a == 2 ? silu_fast(x) : (a ? fmaxf(x, 0.f) : x);
  else return a ? fmaxf(x, 0.f) : x;
}

template <bool SILU>
__global__ void __launch_bounds__(kThreads, 1) tc_chain_kernel(const __grid_constant__ TcChainDesc d, RunPtrs p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  const int S = d.stages;
  const int slot = d.slot_a + d.slot_b;
  const int NS = d.ns;
  uint8_t* wres = smem;
  uint8_t* abuf = smem + d.off_abuf;
  uint8_t* ring = smem + d.off_ring;
  uint8_t* fring = smem + d.off_fring;
  uint8_t* pbuf = smem + d.off_p;
  uint8_t* ones = smem + d.off_ones;
  uint8_t* zeros = smem + d.off_zeros;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + d.off_bars);
  uint64_t* full = bars;                  // [S]
  uint64_t* empty = full + S;             // [S]
  uint64_t* ffull = empty + S;            // [fstages]
  uint64_t* fempty = ffull + 4;           // [fstages]
  uint64_t* acc_full = fempty + 4;        // [NS]
  uint64_t* acc_empty = acc_full + 8;     // [NS]
  uint64_t* p_full = acc_empty + 8;       // [4] (team * 2 + chunk parity)
  uint64_t* p_empty = p_full + 4;         // [4]
  uint64_t* out_full = p_empty + 4;       // [2]
  uint64_t* out_empty = out_full + 2;     // [2]
  uint64_t* wbar = out_empty + 2;
  uint64_t* a_full = wbar + 1;            // [2] A buffers
  uint64_t* a_empty = a_full + 2;         // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(a_empty + 2);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  // constant A operand of the zero-init MMA: K column 0 = 1.0 (bf16), one SW32 atom
  for (int i = threadIdx.x; i < 128 * 2; i += blockDim.x) {
    const int row = i / 2, ch = i % 2;
    uint4 v = make_uint4(0, 0, 0, 0);
    if (ch == swz_chunk(row, 0, 16)) v.x = 0x00003F80u;
    reinterpret_cast<uint4*>(ones)[i] = v;
  }
  for (int i = threadIdx.x; i < 4096 / 16; i += blockDim.x) reinterpret_cast<uint4*>(zeros)[i] = make_uint4(0, 0, 0, 0);
  fence_proxy_async();
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int s = 0; s < 4; ++s) {
      mbar_init(&ffull[s], 1);
      mbar_init(&fempty[s], 1);
      mbar_init(&p_full[s], kTeamArrivals);
      mbar_init(&p_empty[s], 1);
    }
    for (int s = 0; s < 8; ++s) {
      mbar_init(&acc_full[s], 1);
      mbar_init(&acc_empty[s], kTeamArrivals);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&out_full[b], 1);
      mbar_init(&out_empty[b], kTeamArrivals);
    }
    mbar_init(wbar, 1);
    for (int b = 0; b < 2; ++b) {
      mbar_init(&a_full[b], 1);
      mbar_init(&a_empty[b], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  // per-tile programs -> SMEM
  const TcProdOp* prod = d.prod;
  const TcMmaOpD* mprog = d.mma;
  if (d.prog_smem) {
    uint8_t* ps = smem + d.off_prog;
    const int n16 = (d.n_prod * (int)sizeof(TcProdOp) + d.n_mma * (int)sizeof(TcMmaOpD)) / 16;
    const uint4* src = reinterpret_cast<const uint4*>(d.prod);
    for (int i = threadIdx.x; i < n16; i += blockDim.x) reinterpret_cast<uint4*>(ps)[i] = src[i];
    prod = reinterpret_cast<const TcProdOp*>(ps);
    mprog = reinterpret_cast<const TcMmaOpD*>(ps + d.n_prod * sizeof(TcProdOp));
  }
  if (warp == kFWarp) {
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
  const int U = d.units;
#ifdef TEMCO_TRACE
  int tn[kTraceRows] = {0};
#endif
  const bool has_w = d.resident || d.fres;

  // register rebalancing inside the CTA's launch allocation (640 x 96): the role
  // warpgroup (warps 16-19) drops to 40, the four epilogue warpgroups rise to
  // 104 (128*40 + 512*104 <= 640*96); each branch is dominated by its setmaxnreg
  if (warp >= kEpiWarps) {
  asm volatile("setmaxnreg.dec.sync.aligned.u32 40;");
  if (warp == kProdWarp) {
    // ------------------------------------------------------------ TMA producer (A / B ring)
    const char* dbase = reinterpret_cast<const char*>(&d);
    if (has_w && lane == 0) {
      // every resident box once: term atoms of the chunks a term reaches, F atoms
      mbar_expect_tx(wbar, (uint32_t)((d.resident ? d.fbase : 0) + (d.fres ? d.nchunks * d.Np * 128 : 0)));
      if (d.resident) {
        const int nall = d.npc ? d.mt1 : d.n_terms;
        for (int j = 0; j < nall; ++j) {
          const TcTerm& t = d.term[j];
          const int ka_n = t.Rp / t.aw, bb = d.Cc * t.aw * 2;
          for (int c = 0; c < t.nhit; ++c)
            for (int ka = 0; ka < ka_n; ++ka)
              tma_load_2d(wres + t.wres + (c * ka_n + ka) * bb, t.wmap, wbar, ka * t.aw, (t.cfirst + c) * d.Cc);
        }
      }
      if (d.fres)
        for (int c = 0; c < d.nchunks; ++c) tma_load_2d(wres + d.fbase + c * d.Np * 128, d.fmap, wbar, c * 64, 0);
    }
    __syncwarp();
    Ring r{0, 0};
    const int np = d.n_prod, na = d.n_aload;
    int it = 0;
    for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x, ++it) {
      const TileGeo gg = tile_geo(d, tile);
      // the tile's reduced-input atoms, once, into A buffer ab
      const int ab = d.nabuf == 2 ? (it & 1) : 0;
      const int use = d.nabuf == 2 ? (it >> 1) : it;
      mbar_wait(&a_empty[ab], ((uint32_t)use & 1u) ^ 1u);
      mbar_expect_tx_w(&a_full[ab], (uint32_t)d.a_tx);
      uint8_t* ba = abuf + ab * d.abytes;
      for (int i = 0; i < na; ++i) {
        const TcProdOp o = prod[i];
        if (o.kind & PK_A4D)        // (tap-shifted) strided box of the term's input
          tma_load_4d_w(ba + o.dst, dbase + o.amap * 64, &a_full[ab], o.ac, gg.w0 * o.ts + o.dx, gg.h0 * o.ts + o.dy,
                        gg.n0);
        else
          tma_load_2d_w(ba + o.dst, dbase + o.amap * 64, &a_full[ab], o.ac, gg.m0);
      }
      TRACE(0);
      // streamed weights: one ring stage per MMA op
      for (int i = na; i < np; ++i) {
        const TcProdOp o = prod[i];
        mbar_wait(&empty[r.s], r.ph ^ 1);
        mbar_expect_tx_w(&full[r.s], o.bytes);
        tma_load_2d_w(ring + r.s * slot, dbase + o.bmap * 64, &full[r.s], o.bx, o.by);
        r.next(S);
      }
    }
  } else if (warp == kFWarp) {
    // ------------------------------------------------------------ F ring producer (F not resident)
    if (!d.gap && !d.store && !d.fres) {
      Ring r{0, 0};
      for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x)
        for (int c = 0; c < d.nchunks; ++c) {
          mbar_wait(&fempty[r.s], r.ph ^ 1);
          mbar_expect_tx_w(&ffull[r.s], (uint32_t)(d.Np * 128));
          tma_load_2d_w(fring + r.s * d.fslot, d.fmap, &ffull[r.s], c * 64, 0);
          r.next(d.fstages);
        }
    }
  } else if (warp == kMmaWarp) {
    // ------------------------------------------------------------ GEMM1 issuer
    if (has_w) mbar_wait(wbar, 0);
    Ring st{0, 0};
    Ring slr[2] = {{0, 0}, {0, 0}};      // per-team accumulator sub-rings
    const int NST = NS / 2;
    int it = 0;
    const int nm = d.n_mma;
    const uint64_t base16 = smem_u32(smem) >> 4;
    const uint32_t ub = (uint32_t)d.ubuf;
    for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x, ++it) {
      Ring& sl = slr[it & 1];
      const int sbase = (it & 1) * NST;
      const int ab = d.nabuf == 2 ? (it & 1) : 0;
      const int use = d.nabuf == 2 ? (it >> 1) : it;
      mbar_wait(&a_full[ab], (uint32_t)use & 1u);
      TRACE(1);
      tc_fence_after();
      const uint64_t ab16 = (uint64_t)((ab * d.abytes) >> 4);
      for (int i = 0; i < nm; ++i) {
        const TcMmaOpD o = mprog[i];
        const uint32_t f = o.flags;
        if (f & MF_ACC_WAIT) {
          mbar_wait(&acc_empty[sbase + sl.s], sl.ph ^ 1);
          TRACE(2);
          tc_fence_after();
        }
        if (f & MF_SW) {
          mbar_wait(&full[st.s], st.ph);
          tc_fence_after();
        }
        const uint64_t st16 = (uint64_t)((st.s * slot) >> 4);
        const uint64_t ad = o.adesc + base16 + ((f & MF_AT) ? ab16 : 0);
        const uint64_t bd = o.bdesc + base16 + ((f & MF_SB) ? st16 : 0);
        const uint32_t dt = tbase + (uint32_t)(sbase + sl.s) * ub + o.tmem;
        if (!(d.exp & 2)) {
          mma_bf16_w(dt, ad, bd, o.idesc, (f & MF_ZERO) ? 0u : 1u);
          for (int k = 1; k < o.nk; ++k) mma_bf16_w(dt, ad + 2 * k, bd + 2 * k, o.idesc, 1u);
        }
        if (f & MF_SD) {
          mma_commit_w(&empty[st.s]);
          st.next(S);
        }
        if (f & MF_ACC_COMMIT) {
          mma_commit_w(&acc_full[sbase + sl.s]);
          TRACE(3);
          sl.next(NST);
        }
      }
      mma_commit_w(&a_empty[ab]);   // the tile's A buffer is free once its MMAs complete
    }
  } else if (warp == kG2Warp) {
    // ------------------------------------------------------------ GEMM2 issuer: out += P_c F_c^T
    if (!d.gap && !d.store) {
      if (d.fres) mbar_wait(wbar, 0);
      Ring fr{0, 0};
      uint32_t pph = 0;                 // phase bits of the 4 P buffers
      const uint32_t idesc2 = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(d.Np >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
      const uint64_t pdesc0 = umma_desc(smem_u32(pbuf));
      int it = 0;
      for (int tile = blockIdx.x; tile < d.ntiles; tile += gridDim.x, ++it) {
        const int team = it & 1;
        // output buffer: one per team (no == 2) or shared (no == 1); out_full /
        // out_empty barriers are per team so every wait has a single in-order party
        const int ob = d.no == 2 ? team : 0;
        if (d.no == 2) {
          mbar_wait(&out_empty[team], (((uint32_t)it >> 1) & 1u) ^ 1u);
        } else if (it > 0) {
          mbar_wait(&out_empty[(it - 1) & 1], ((uint32_t)(it - 1) >> 1) & 1u);
        }
        TRACE(11);
        tc_fence_after();
        const uint32_t dt = tbase + (uint32_t)(d.out_col + ob * d.Np);
        int cp = 0;                     // chunk index among the tile's finished chunks
        for (int u = 0; u < U; ++u) {
          const Unit un = unit_at(d, u);
          if (!un.last) continue;
          const int pb = team * 2 + (cp & 1);
          mbar_wait(&p_full[pb], (pph >> pb) & 1u);
          TRACE(7);
          pph ^= 1u << pb;
          tc_fence_after();
          uint64_t bdesc;
          if (d.fres) {
            bdesc = umma_desc(smem_u32(wres + d.fbase + un.c * d.Np * 128));
          } else {
            mbar_wait(&ffull[fr.s], fr.ph);
            tc_fence_after();
            bdesc = umma_desc(smem_u32(fring + fr.s * d.fslot));
          }
          const uint64_t adesc = pdesc0 + (uint64_t)((pb * 16384) >> 4);
#pragma unroll
          for (int k = 0; k < 4; ++k) mma_bf16_w(dt, adesc + 2 * k, bdesc + 2 * k, idesc2, (cp | k) ? 1u : 0u);
          mma_commit_w(&p_empty[pb]);
          TRACE(8);
          if (!d.fres) {
            mma_commit_w(&fempty[fr.s]);
            fr.next(d.fstages);
          }
          ++cp;
        }
        mma_commit_w(&out_full[team]);
      }
    }
  }
  } else {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 104;");
    // ------------------------------------------------------------ epilogue teams
    // team k takes the CTA's tiles k, k+2, ...; warp tw of a team: TMEM lane
    // quarter q = warp % 4 (pixel rows 32q..32q+31), column half h (32 of the unit's 64)
    const int team = warp / kTeamWarps, tw = warp % kTeamWarps;
    const int q = warp & 3, h = tw >> 2;
    const int row = q * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    const int c_lo = h * 32;
    __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.arena + d.y.off);
    uint32_t pph = 0;
    int it = team;
    const int NST = NS / 2, sbase = team * NST;
    Ring sl{0, 0};                        // this team's accumulator sub-ring
    for (int tile = blockIdx.x + team * gridDim.x; tile < d.ntiles; tile += 2 * gridDim.x, it += 2) {
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
      // accumulator slot of this tile's first unit-level
      float t[32];   // running level value t_l (pooled units: running max / sum over taps)
      int cp = 0;
      for (int u = 0; u < U; ++u) {
        const Unit un = unit_at(d, u);
        const int col0 = un.c * d.Cc + c_lo;           // first restored channel of this thread
        const int nl = un.pooled ? 1 : d.n_levels;
        for (int l = 0; l < nl; ++l) {
          const bool last = un.last && l == nl - 1;
          mbar_wait(&acc_full[sbase + sl.s], sl.ph);
          if (warp == 0) TRACE(4);
          if (warp == kTeamWarps) TRACE(10);
          tc_fence_after();
          const uint32_t ta = tbase + lane_off + (uint32_t)((sbase + sl.s) * d.ubuf + c_lo);
          if (un.pooled) {
            // pooled member: fold this unit's taps (max of the raw accumulators, or
            // sum of act(acc + b)) into the running value
            if (un.tg == 0) {
#pragma unroll
              for (int i = 0; i < 32; ++i) t[i] = d.mpool == 1 ? -INFINITY : 0.f;
            }
            const float4* b4 = reinterpret_cast<const float4*>(p.params + d.mbias + col0);
            for (int r = 0; r < un.nt; ++r) {
              const int tap = un.tg * d.tpu + r;
              const int hi = ho * d.ms - d.mp + tap / d.mk, wi = wo * d.ms - d.mp + tap % d.mk;
              const bool valid = hi >= 0 && hi < d.mHin && wi >= 0 && wi < d.mWin;
              uint32_t v[32];
              tmem_ld32(ta + r * d.Cc, v);
              tmem_wait_ld();
              if (d.mpool == 1 && !(SILU && d.mrelu == 2)) {
                // monotone activation: max of the raw accumulators, bias + act after the pool
                if (valid) {
#pragma unroll
                  for (int i = 0; i < 32; ++i) t[i] = fmaxf(t[i], __uint_as_float(v[i]));
                }
              } else if (d.mpool == 1) {
                // SiLU is not monotone (minimum near -1.28): max over act(acc + b) per tap
                if (valid) {
#pragma unroll
                  for (int i4 = 0; i4 < 8; ++i4) {
                    const float4 bb = __ldg(b4 + i4);
                    const float bq[4] = {bb.x, bb.y, bb.z, bb.w};
#pragma unroll
                    for (int k = 0; k < 4; ++k)
                      t[4 * i4 + k] = fmaxf(t[4 * i4 + k], act_m<SILU>(__uint_as_float(v[4 * i4 + k]) + bq[k], d.mrelu));
                  }
                }
              } else {
#pragma unroll
                for (int i4 = 0; i4 < 8; ++i4) {
                  const float4 bb = __ldg(b4 + i4);
                  const float bq[4] = {bb.x, bb.y, bb.z, bb.w};
#pragma unroll
                  for (int k = 0; k < 4; ++k) {
                    const float z = __uint_as_float(v[4 * i4 + k]) + bq[k];
                    t[4 * i4 + k] += act_m<SILU>(z, d.mrelu);
                  }
                }
              }
            }
            tc_fence_before();
            warp_arrive(&acc_empty[sbase + sl.s]);
            sl.next(NST);
            if (!un.last) continue;
            // pooled value (+ member bias, act, for max), + post-pool shift -> t
            const float4* p4 = reinterpret_cast<const float4*>(p.params + (d.post >= 0 ? d.post : d.mbias) + col0);
            const float pscale = d.post >= 0 ? 1.f : 0.f;
            const float sc = d.mpool == 2 ? 1.f / (float)d.mtaps : 1.f;
            const float4* s4 = reinterpret_cast<const float4*>(p.params + (d.postsc >= 0 ? d.postsc : d.mbias) + col0);
#pragma unroll
            for (int i4 = 0; i4 < 8; ++i4) {
              const float4 bb = __ldg(b4 + i4), pp = __ldg(p4 + i4);
              const float4 ss = d.postsc >= 0 ? __ldg(s4 + i4) : make_float4(1.f, 1.f, 1.f, 1.f);
              const float bq[4] = {bb.x, bb.y, bb.z, bb.w}, pq[4] = {pp.x, pp.y, pp.z, pp.w};
              const float sq[4] = {ss.x, ss.y, ss.z, ss.w};
#pragma unroll
              for (int k = 0; k < 4; ++k) {
                const int i = 4 * i4 + k;
                float z = t[i] * sc;
                if (d.mpool == 1 && !(SILU && d.mrelu == 2)) {
                  z += bq[k];
                  z = act_m<SILU>(z, d.mrelu);
                }
                t[i] = z * sq[k] + pscale * pq[k];
              }
            }
          } else if (d.exp & 1) {
            warp_arrive(&acc_empty[sbase + sl.s]);
            sl.next(NST);
          } else {
            uint32_t v[32];
            tmem_ld32(ta, v);
            const float4* b4 = reinterpret_cast<const float4*>(p.params + d.lbias[l] + col0);
            tmem_wait_ld();
            tc_fence_before();
            warp_arrive(&acc_empty[sbase + sl.s]);
            if (warp == 0) TRACE(5);
            sl.next(NST);
#pragma unroll
            for (int i4 = 0; i4 < 8; ++i4) {
              const float4 bb = __ldg(b4 + i4);
              const float bq[4] = {bb.x, bb.y, bb.z, bb.w};
#pragma unroll
              for (int k = 0; k < 4; ++k) {
                const int i = 4 * i4 + k;
                const float z = __uint_as_float(v[i]) + bq[k];
                t[i] = l == 0 ? z : z + t[i];
              }
            }
          }
          const int act = d.relu[un.pooled ? 0 : l];
          if (SILU && act == 2) {   // SiLU level: applied in place, then the no-activation path
#pragma unroll
            for (int i = 0; i < 32; ++i) t[i] = silu_fast(t[i]);
          }
          const bool relu = SILU ? act == 1 : act != 0;
          if (!last) {
            if (relu) {
#pragma unroll
              for (int i = 0; i < 32; ++i) t[i] = fmaxf(t[i], 0.f);
            }
            continue;
          }
          if (d.gap) {
            // GAP root: per-image column means; tiles hold whole images so the
            // summation order is fixed (deterministic, batch-invariant)
            float* red = reinterpret_cast<float*>(pbuf + (team * 2 + h) * 16384);
#pragma unroll
            for (int i = 0; i < 32; ++i) red[row * 32 + ((i + row) & 31)] = relu ? fmaxf(t[i], 0.f) : t[i];
            const int bar_id = 1 + team * 2 + h;
            asm volatile("bar.sync %0, 128;" ::"r"(bar_id) : "memory");
            for (int idx = row; idx < d.ipt * 32; idx += 128) {
              const int ii = idx / 32, col = idx % 32;
              const int n = tile * d.ipt + ii;
              float acc = 0.f;
              for (int rr = ii * d.hw; rr < (ii + 1) * d.hw; ++rr) acc += red[rr * 32 + ((col + rr) & 31)];
              const int cg = col0 + col;
              if (n < d.nimg && cg < d.C) y[(int64_t)n * d.C + cg] = __float2bfloat16_rn(acc / (float)d.hw);
            }
            asm volatile("bar.sync %0, 128;" ::"r"(bar_id) : "memory");
            continue;
          }
          if (d.store) {
            // store root: the restored value itself, bf16 NHWC [npix, C]
            if (mvalid) {
              uint4* dst = reinterpret_cast<uint4*>(y + m * d.C + col0);
#pragma unroll
              for (int qq = 0; qq < 4; ++qq) {
                uint4 pk;
                pk.x = relu ? pack_bf16_relu(t[8 * qq + 0], t[8 * qq + 1]) : pack_bf16(t[8 * qq + 0], t[8 * qq + 1]);
                pk.y = relu ? pack_bf16_relu(t[8 * qq + 2], t[8 * qq + 3]) : pack_bf16(t[8 * qq + 2], t[8 * qq + 3]);
                pk.z = relu ? pack_bf16_relu(t[8 * qq + 4], t[8 * qq + 5]) : pack_bf16(t[8 * qq + 4], t[8 * qq + 5]);
                pk.w = relu ? pack_bf16_relu(t[8 * qq + 6], t[8 * qq + 7]) : pack_bf16(t[8 * qq + 6], t[8 * qq + 7]);
                dst[qq] = pk;
              }
            }
            continue;
          }
          // last level: P = bf16 act(x) -> SMEM (one SW128 K-major atom per 64-channel unit)
          const int pb = team * 2 + (cp & 1);
          mbar_wait(&p_empty[pb], ((pph >> pb) & 1u) ^ 1u);
          pph ^= 1u << pb;
          uint8_t* prow = pbuf + pb * 16384 + row * 128;
#pragma unroll
          for (int qq = 0; qq < 4; ++qq) {
            uint4 pk;
            if (relu) {
              pk.x = pack_bf16_relu(t[8 * qq + 0], t[8 * qq + 1]);
              pk.y = pack_bf16_relu(t[8 * qq + 2], t[8 * qq + 3]);
              pk.z = pack_bf16_relu(t[8 * qq + 4], t[8 * qq + 5]);
              pk.w = pack_bf16_relu(t[8 * qq + 6], t[8 * qq + 7]);
            } else {
              pk.x = pack_bf16(t[8 * qq + 0], t[8 * qq + 1]);
              pk.y = pack_bf16(t[8 * qq + 2], t[8 * qq + 3]);
              pk.z = pack_bf16(t[8 * qq + 4], t[8 * qq + 5]);
              pk.w = pack_bf16(t[8 * qq + 6], t[8 * qq + 7]);
            }
            const int ch = h * 4 + qq;
            *reinterpret_cast<uint4*>(prow + ((ch ^ (row & 7)) * 16)) = pk;
          }
          fence_proxy_async();
          warp_arrive(&p_full[pb]);
          if (warp == 0) TRACE(6);
          ++cp;
        }
      }
      if (d.gap || d.store) continue;
      // output epilogue: column groups of 8 split between the two column halves
      const int ob = d.no == 2 ? team : 0;
      mbar_wait(&out_full[team], (uint32_t)(it >> 1) & 1u);
      if (warp == 0) TRACE(9);
      tc_fence_after();
      const int ng = d.Np / 8, gh = (ng + 1) / 2;
      const int gend = min(ng, (h + 1) * gh);
      const uint32_t to = tbase + lane_off + (uint32_t)(d.out_col + ob * d.Np);
      __nv_bfloat16* yrow = y + m * d.Nout;
      const int gvalid = mvalid ? min(gend, d.Nout / 8) : 0;
      for (int g0 = h * gh; g0 < gend; g0 += 2) {
        uint32_t v0[8], v1[8];
        tmem_ld8(to + g0 * 8, v0);
        if (g0 + 1 < gend) tmem_ld8(to + (g0 + 1) * 8, v1);
        tmem_wait_ld();
        if (g0 < gvalid) {
          uint4 pk;
          pk.x = pack_bf16(__uint_as_float(v0[0]), __uint_as_float(v0[1]));
          pk.y = pack_bf16(__uint_as_float(v0[2]), __uint_as_float(v0[3]));
          pk.z = pack_bf16(__uint_as_float(v0[4]), __uint_as_float(v0[5]));
          pk.w = pack_bf16(__uint_as_float(v0[6]), __uint_as_float(v0[7]));
          *reinterpret_cast<uint4*>(yrow + g0 * 8) = pk;
        }
        if (g0 + 1 < gvalid) {
          uint4 pk;
          pk.x = pack_bf16(__uint_as_float(v1[0]), __uint_as_float(v1[1]));
          pk.y = pack_bf16(__uint_as_float(v1[2]), __uint_as_float(v1[3]));
          pk.z = pack_bf16(__uint_as_float(v1[4]), __uint_as_float(v1[5]));
          pk.w = pack_bf16(__uint_as_float(v1[6]), __uint_as_float(v1[7]));
          *reinterpret_cast<uint4*>(yrow + (g0 + 1) * 8) = pk;
        }
      }
      tc_fence_before();
      warp_arrive(&out_empty[team]);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == kFWarp) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tbase), "r"(d.tmem_cols));
  }
}

}  // namespace

#ifdef TEMCO_TRACE
extern "C" void temco_debug_trace(long long* out) {
  cudaMemcpyFromSymbol(out, g_trace, sizeof(g_trace));
  void* p = nullptr;
  cudaGetSymbolAddress(&p, g_trace);
  cudaMemset(p, 0, sizeof(g_trace));
}
#endif

// diagnostics: registers, max threads per block, static / max dynamic SMEM of the chain kernel
extern "C" int temco_debug_tc_attrs(int* out) {
  cudaFuncAttributes a;
  const cudaError_t e = cudaFuncGetAttributes(&a, tc_chain_kernel<false>);
  out[0] = a.numRegs;
  out[1] = a.maxThreadsPerBlock;
  out[2] = (int)a.sharedSizeBytes;
  out[3] = a.maxDynamicSharedSizeBytes;
  out[4] = (int)a.localSizeBytes;
  return (int)e;
}

void launch_tc_chain(const TcChainDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s) {
  (void)tcw;
  static bool configured = false;
  static int sms = 0;
  if (!configured) {
    cudaFuncSetAttribute(tc_chain_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    cudaFuncSetAttribute(tc_chain_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    configured = true;
  }
  const int grid = std::min(d.ntiles, sms > 0 ? sms : 148);
  // >= 114 KB of shared memory keeps one CTA per SM (each owns all 512 TMEM columns)
  const bool silu = d.mrelu == 2 || std::any_of(d.relu, d.relu + d.n_levels, [](int32_t a) { return a == 2; });
  launch_pdl(silu ? tc_chain_kernel<true> : tc_chain_kernel<false>, dim3(grid), dim3(kThreads),
             std::max(d.smem_bytes, 116 * 1024), s, d, p);
}

}  // namespace temco
