// Group -> "level chain" parser shared by the tcgen05 (kernels_tc.cu) and the
// mma.sync (kernels_mma.cu) lowerings (reading R12):
//   t_l = act_l( sum_{j in l} diag(scale_j) L_j r_j + b_l + t_{l-1} )
// BN layers fold into per-row scales and the level bias, adds merge terms
// (P:L333), concats place terms at channel offsets (Fig. 9a).
#pragma once

#include <cmath>
#include <set>
#include <vector>

#include "planner.h"

namespace temco {
namespace chainp {

struct PTerm {
  int lconv;
  std::vector<double> scale;   // per row of the lconv output
  int c0;
};

struct PLevel {
  std::vector<PTerm> terms;
  std::vector<double> bias;
  bool relu = false;
};

struct ChainParser {
  const IR& ir;
  std::set<int> members;
  int C;
  std::set<int> visited;
  int H, W;

  bool chain(int v, std::vector<PLevel>& out) {
    if (!members.count(v)) return false;
    visited.insert(v);
    if (ir.nodes[v].op == OP_RELU) {
      if (!pre(ir.oin[v][0], out)) return false;
      out.back().relu = true;
      return true;
    }
    return pre(v, out);
  }

  bool pre(int v, std::vector<PLevel>& out) {
    PLevel L;
    L.bias.assign(C, 0.0);
    std::vector<PLevel> prev;
    if (!contribute(v, nullptr, 0, L, prev)) return false;
    if (L.terms.empty()) return false;
    out = prev;
    out.push_back(L);
    return true;
  }

  bool contribute(int v, const std::vector<double>* sc, int c0, PLevel& L, std::vector<PLevel>& prev) {
    if (!members.count(v)) return false;   // external full tensor: not on this kernel
    visited.insert(v);
    const Node& n = ir.nodes[v];
    if (n.H != H || n.W != W) return false;
    if (n.role == ROLE_LCONV) {
      PTerm t;
      t.lconv = v;
      t.c0 = c0;
      t.scale = sc ? *sc : std::vector<double>(n.C, 1.0);
      if (n.b)
        for (int c = 0; c < n.C; ++c) L.bias[c0 + c] += t.scale[c] * (*n.b)[c];
      L.terms.push_back(std::move(t));
      return true;
    }
    switch (n.op) {
      case OP_BN: {
        std::vector<double> s(n.C);
        for (int c = 0; c < n.C; ++c) {
          double k = (double)(*n.bn_g)[c] / std::sqrt((double)(*n.bn_v)[c] + (double)n.eps);
          double sh = (double)(*n.bn_b)[c] - (double)(*n.bn_m)[c] * k;
          double outer = sc ? (*sc)[c] : 1.0;
          s[c] = outer * k;
          L.bias[c0 + c] += outer * sh;
        }
        return contribute(ir.oin[v][0], &s, c0, L, prev);
      }
      case OP_ADD:
        for (int x : ir.oin[v])
          if (!contribute(x, sc, c0, L, prev)) return false;
        return true;
      case OP_CONCAT: {
        int off = 0;
        for (int x : ir.oin[v]) {
          const int cx = ir.nodes[x].C;
          std::vector<double> s2;
          if (sc) s2.assign(sc->begin() + off, sc->begin() + off + cx);
          if (!contribute(x, sc ? &s2 : nullptr, c0 + off, L, prev)) return false;
          off += cx;
        }
        return true;
      }
      case OP_RELU: {
        // a previous chain value t_{l-1}: unit scale, full width, at most one
        if (sc || c0 != 0 || n.C != C || !prev.empty()) return false;
        return chain(v, prev);
      }
      default:
        return false;
    }
  }
};


}  // namespace chainp
}  // namespace temco
