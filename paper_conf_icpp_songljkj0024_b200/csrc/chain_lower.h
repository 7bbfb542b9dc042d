// Host-side lowering shared by the two one-CTA tcgen05 chain kernels (kernels_tc.cu: SMEM-staged
// levels; kernels_tc_wide.cu: TMEM-resident levels): the bf16 / fp32 parameter pools, the tile
// geometry of a parsed chain (chain_parse.h) and the packing of one restore term.  Both TcChainDesc
// types carry the same geometry and term fields; only the chunk width Cc is chosen by the caller.
#pragma once

#include <algorithm>
#include <cstdint>
#include <cstring>
#include <map>
#include <vector>

#include "chain_parse.h"
#include "device.h"
#include "planner.h"

namespace temco {
namespace chainl {

inline uint16_t to_bf16(float f) {
  uint32_t u;
  memcpy(&u, &f, 4);
  u += 0x7FFF + ((u >> 16) & 1);
  return (uint16_t)(u >> 16);
}

inline int64_t push_bf16(std::vector<uint16_t>& pool, const std::vector<float>& v) {
  while (pool.size() % 512) pool.push_back(0);   // 1024-byte aligned blocks (TMA base alignment)
  int64_t off = (int64_t)pool.size();
  for (float f : v) pool.push_back(to_bf16(f));
  return off;
}

// fp32 vector padded with zeros to n entries, 16-byte aligned in the params pool
inline int64_t push_f32(std::vector<float>& params, const std::vector<double>& v, int n) {
  while (params.size() % 4) params.push_back(0.f);
  const int64_t off = (int64_t)params.size();
  for (int i = 0; i < n; ++i) params.push_back(i < (int)v.size() ? (float)v[i] : 0.f);
  return off;
}

// tiles of the chain's output pixels: 128-row tiles; GAP roots take whole images per tile;
// chains with tap-shifted terms ("spatial") take tw x th x tn boxes.  d.C / d.Cc set by the caller.
template <class D>
bool tile_geometry(D& d, const IR& ir, const Node& tn, int Nout, bool gap, bool spatial, const Loc& y, int n_levels) {
  d.Cpad = (d.C + d.Cc - 1) / d.Cc * d.Cc;
  d.nchunks = d.Cpad / d.Cc;
  d.Nout = Nout;
  d.Np = (Nout + 15) / 16 * 16;
  d.npix = (int64_t)ir.batch * tn.H * tn.W;
  d.nimg = ir.batch;
  d.gap = gap ? 1 : 0;
  d.hw = tn.H * tn.W;
  d.Ho = tn.H;
  d.Wo = tn.W;
  d.spatial = spatial ? 1 : 0;
  d.post = -1;
  d.postsc = -1;
  if (d.spatial) {
    d.tw = std::min(tn.W, 128);
    d.th = std::min(tn.H, 128 / d.tw);
    d.tn = (d.th == tn.H && d.tw == tn.W) ? std::max(1, std::min(ir.batch, 128 / (tn.H * tn.W))) : 1;
    d.nwb = (tn.W + d.tw - 1) / d.tw;
    d.nhb = (tn.H + d.th - 1) / d.th;
    d.nnb = (ir.batch + d.tn - 1) / d.tn;
    d.mused = d.tw * d.th * d.tn;
    d.ntiles = d.nnb * d.nhb * d.nwb;
    d.rows_per_tile = 128;
    if (gap) {
      if (d.th != tn.H || d.tw != tn.W) return false;    // GAP needs whole images per tile
      d.ipt = d.tn;
    }
  } else if (gap) {
    d.ipt = 128 / d.hw;
    d.rows_per_tile = d.ipt * d.hw;
    d.ntiles = (ir.batch + d.ipt - 1) / d.ipt;
  } else {
    d.rows_per_tile = 128;
    d.ntiles = (int)((d.npix + 127) / 128);
  }
  d.y = y;
  d.n_levels = n_levels;
  return true;
}

// one restore term (an lconv over reduced input r): BN-folded Lhat rows at its channel range,
// bf16 [Cpad][Rw]; accumulates the algorithmic FLOPs / bytes
template <class D, class T>
bool add_term(D& d, T& term, const IR& ir, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
              const chainp::PTerm& t, int64_t& flops, int64_t& bytes) {
  const Node& lc = ir.nodes[t.lconv];
  const int r = ir.oin[t.lconv][0];
  const Node& rn = ir.nodes[r];
  const int R = rn.C;
  term.r = loc.at(r);
  term.R = R;
  term.aw = R <= 16 ? 16 : R <= 32 ? 32 : 64;      // box width ~ rank: no mostly-OOB boxes
  term.Rp = (R + term.aw - 1) / term.aw * term.aw;
  term.Rw = (R + 7) / 8 * 8;
  term.c0 = t.c0;
  term.C = lc.C;
  term.Hin = rn.H;
  term.Win = rn.W;
  term.tk = t.tk;
  term.ts = t.ts;
  term.tp = t.tp;
  term.cfirst = t.c0 / d.Cc;
  term.nhit = (t.c0 + lc.C - 1) / d.Cc - term.cfirst + 1;
  std::vector<float> w((size_t)d.Cpad * term.Rw, 0.f);
  for (int c = 0; c < lc.C; ++c)
    for (int k = 0; k < R; ++k) w[(size_t)(t.c0 + c) * term.Rw + k] = (float)(t.scale[c] * (*lc.w)[(size_t)c * R + k]);
  term.w = push_bf16(tcw, w);
  const int64_t in_pix = (int64_t)ir.batch * rn.H * rn.W;
  flops += in_pix * 2LL * lc.C * R;
  bytes += in_pix * 2LL * R;
  return !(d.spatial && (d.tw * term.ts > 256 || d.th * term.ts > 256));
}

}  // namespace chainl
}  // namespace temco
