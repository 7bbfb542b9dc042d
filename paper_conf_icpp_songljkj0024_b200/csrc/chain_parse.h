// Group -> "level chain" parser shared by the tcgen05 (kernels_tc.cu) and the
// mma.sync (kernels_mma.cu) lowerings (reading R12):
//   t_l = act_l( sum_{j in l} diag(scale_j) L_j r_j + b_l + t_{l-1} )
// BN layers fold into per-row scales and the level bias, adds merge terms
// (P:L333), concats place terms at channel offsets (Fig. 9a).
//
// Pooled members (Listing 1 with p >= 2) inside a level:
//  * avgpool over a *linear* member (e.g. DenseNet's transition output
//    avgpool(lconv(r))) is linear, avgpool(L r + b) = L avgpool(r) + b, so its
//    terms become "tap-accumulate" terms (k*k tap-shifted reads of r summed
//    into the same accumulator, weights / k^2);
//  * any other pool (max, or over a ReLU) becomes a PMember evaluated per tap:
//    pool_tap( act(sum scale L r + b) ), then the level's own bias (the post-BN
//    shift) and activation.  A BN after a max-pool folds through it only for
//    positive scales (max(s x) = s max(x), s > 0); otherwise the parse fails.
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
  int tk = 1, ts = 1, tp = 0;  // tap-accumulate (folded avg pool): k x k window, stride, pad
};

struct PMember {               // pooled non-linear member (per-tap epilogue)
  int c0 = 0, C = 0;
  int kind = 1;                // 1 max, 2 avg
  int k = 1, s = 1, p = 0;
  int Hin = 0, Win = 0;
  std::vector<PTerm> terms;
  std::vector<double> bias;    // member bias (size C), scaled
  bool relu = false;
  bool silu = false;           // only with allow_silu
  std::vector<double> post_scale;   // SiLU member: the post-pool BN scale, applied after the pool
};

struct PLevel {
  std::vector<PTerm> terms;
  std::vector<double> bias;
  bool relu = false;
  bool silu = false;           // SiLU activation of the level, only with allow_silu
  std::vector<PMember> pm;
  // only with allow_member_act: per-channel activation of activated concat members
  // (UNet decoder: concat(relu(bn(lconv(skip))), lconv(up-conv))); -1 = the level's own
  // activation, 1 ReLU, 2 SiLU, 0 none.  Empty: every channel takes the level activation.
  std::vector<int> act_ch;
};

struct ChainParser {
  const IR& ir;
  std::set<int> members;
  int C;
  std::set<int> visited;
  int H, W;
  bool allow_silu = false;     // set by lowerers whose kernels apply PLevel::silu
  bool allow_member_act = false;   // set by lowerers whose kernels apply PLevel::act_ch

  bool chain(int v, std::vector<PLevel>& out) {
    if (!members.count(v)) return false;
    visited.insert(v);
    const int op = ir.nodes[v].op;
    if (op == OP_RELU || (allow_silu && op == OP_SILU)) {
      if (!pre(ir.oin[v][0], out)) return false;
      (op == OP_RELU ? out.back().relu : out.back().silu) = true;
      return true;
    }
    return pre(v, out);
  }

  bool pre(int v, std::vector<PLevel>& out) {
    PLevel L;
    L.bias.assign(C, 0.0);
    std::vector<PLevel> prev;
    if (!contribute(v, nullptr, 0, L, prev)) return false;
    if (L.terms.empty() && L.pm.empty()) return false;
    out = prev;
    out.push_back(L);
    return true;
  }

  // linear sub-expression (lconv / bn / add) at resolution (h, w): terms + bias
  bool linear(int v, const std::vector<double>* sc, int c0, int h, int w, std::vector<PTerm>& terms,
              std::vector<double>& bias, int bias_off) {
    if (!members.count(v)) return false;
    visited.insert(v);
    const Node& n = ir.nodes[v];
    if (n.H != h || n.W != w) return false;
    if (n.role == ROLE_LCONV) {
      PTerm t;
      t.lconv = v;
      t.c0 = c0;
      t.scale = sc ? *sc : std::vector<double>(n.C, 1.0);
      if (n.b)
        for (int c = 0; c < n.C; ++c) bias[bias_off + c] += t.scale[c] * (*n.b)[c];
      terms.push_back(std::move(t));
      return true;
    }
    if (n.op == OP_BN) {
      std::vector<double> s(n.C);
      for (int c = 0; c < n.C; ++c) {
        double k = (double)(*n.bn_g)[c] / std::sqrt((double)(*n.bn_v)[c] + (double)n.eps);
        double sh = (double)(*n.bn_b)[c] - (double)(*n.bn_m)[c] * k;
        double outer = sc ? (*sc)[c] : 1.0;
        s[c] = outer * k;
        bias[bias_off + c] += outer * sh;
      }
      return linear(ir.oin[v][0], &s, c0, h, w, terms, bias, bias_off);
    }
    if (n.op == OP_ADD) {
      for (int x : ir.oin[v])
        if (!linear(x, sc, c0, h, w, terms, bias, bias_off)) return false;
      return true;
    }
    return false;
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
      case OP_SILU:
        if (!allow_silu) return false;
        [[fallthrough]];
      case OP_RELU: {
        // a previous chain value t_{l-1}: unit scale, full width, at most one
        if (!(sc || c0 != 0 || n.C != C || !prev.empty())) return chain(v, prev);
        // an activated member of a concat (channels [c0, c0 + n.C)): act(linear), its own
        // terms and bias inside this level, the activation recorded per channel
        if (!allow_member_act || sc || (c0 == 0 && n.C == C)) return false;
        std::vector<PTerm> terms;
        std::vector<double> b(n.C, 0.0);
        if (!linear(ir.oin[v][0], nullptr, c0, n.H, n.W, terms, b, 0)) return false;
        for (PTerm& t : terms) L.terms.push_back(std::move(t));
        for (int c = 0; c < n.C; ++c) L.bias[c0 + c] += b[c];
        if (L.act_ch.empty()) L.act_ch.assign(C, -1);
        for (int c = 0; c < n.C; ++c) L.act_ch[c0 + c] = n.op == OP_RELU ? 1 : 2;
        return true;
      }
      case OP_MAXPOOL:
      case OP_AVGPOOL: {
        const int u = ir.oin[v][0];
        const Node& un = ir.nodes[u];
        // avg pool over a linear member: tap-accumulate terms (weights / k^2)
        if (n.op == OP_AVGPOOL && ir.nodes[u].op != OP_RELU) {
          std::vector<PTerm> terms;
          std::vector<double> bias(n.C, 0.0);
          std::set<int> saved = visited;
          if (linear(u, sc, c0, un.H, un.W, terms, bias, 0)) {
            const double inv = 1.0 / (n.kh * n.kw);
            for (PTerm& t : terms) {
              for (double& x : t.scale) x *= inv;
              t.tk = n.kh;
              t.ts = n.sh;
              t.tp = 0;
              L.terms.push_back(t);
            }
            for (int c = 0; c < n.C; ++c) L.bias[c0 + c] += bias[c];
            visited.insert(v);
            return true;
          }
          visited = saved;
        }
        // non-linear pooled member: act(sum scale L r + b) per tap, then pool
        if (sc)
          for (double x : *sc)
            if (!(x > 0.0)) return false;
        PMember m;
        m.c0 = c0;
        m.C = n.C;
        m.kind = n.op == OP_MAXPOOL ? 1 : 2;
        m.k = n.kh;
        m.s = n.sh;
        m.p = n.ph;
        m.Hin = un.H;
        m.Win = un.W;
        m.bias.assign(n.C, 0.0);
        int lin = u;
        if (un.op == OP_RELU || (allow_silu && un.op == OP_SILU)) {
          if (!members.count(u)) return false;
          visited.insert(u);
          (un.op == OP_RELU ? m.relu : m.silu) = true;
          lin = ir.oin[u][0];
        }
        // a post-pool scale s folds into the member only through a positively
        // homogeneous activation (relu(s y) = s relu(y), s > 0); SiLU is not, so
        // its member keeps s aside: s * pool(silu(L r + b)) (+ the level shift)
        const bool keep_scale = m.silu && sc;
        if (keep_scale) m.post_scale = *sc;
        if (!linear(lin, keep_scale ? nullptr : sc, c0, un.H, un.W, m.terms, m.bias, 0)) return false;
        L.pm.push_back(std::move(m));
        return true;
      }
      default:
        return false;
    }
  }
};

}  // namespace chainp
}  // namespace temco
