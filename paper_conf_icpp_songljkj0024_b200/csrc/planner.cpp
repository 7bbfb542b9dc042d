// TeMCO host planner (see planner.h).  Citations are PAPER.md lines (P:L…);
// readings R1..R27 are the DESIGN.md register.
#include "planner.h"

#include <algorithm>
#include <numeric>
#include <set>
#include <tuple>
#include <sstream>

namespace temco {

const char* op_name(Op op) {
  switch (op) {
    case OP_INPUT: return "input";
    case OP_CONV: return "conv";
    case OP_BN: return "bn";
    case OP_RELU: return "relu";
    case OP_SILU: return "silu";
    case OP_ADD: return "add";
    case OP_CONCAT: return "concat";
    case OP_MAXPOOL: return "maxpool";
    case OP_AVGPOOL: return "avgpool";
    case OP_GAP: return "gap";
    case OP_LINEAR: return "linear";
    case OP_CONVT: return "convt";
  }
  return "?";
}

const char* role_name(Role r) {
  switch (r) {
    case ROLE_FCONV: return "fconv";
    case ROLE_CORE: return "core";
    case ROLE_LCONV: return "lconv";
    default: return "";
  }
}

namespace {

Buf copy_buf(const float* p, size_t n) {
  if (!p) return nullptr;
  return std::make_shared<const std::vector<float>>(p, p + n);
}

bool is_lconv(const Node& n) { return n.role == ROLE_LCONV; }     // IsLConv, reading R7

bool recurse_op(Op op) {   // FindReduced walks through these (reading R6)
  return op == OP_BN || op == OP_RELU || op == OP_SILU || op == OP_ADD || op == OP_CONCAT || op == OP_MAXPOOL ||
         op == OP_AVGPOOL;
}

bool absorbable(const Node& n) {   // fusion grouping, reading R12
  return recurse_op(n.op) || is_lconv(n);
}

struct Fail {
  temco_status st;
  std::string msg;
};

[[noreturn]] void fail(temco_status st, const std::string& m) { throw Fail{st, m}; }

// ---------------------------------------------------------------------------
// validation + O1 expansion (Eq. (2); readings R15-R17)
// ---------------------------------------------------------------------------
void expand(const temco_layer* layers, int n_layers, const temco_decomp* decomps, int n_decomps,
            const temco_edge* edges, int n_edges, const temco_config& cfg, bool bf16, IR& ir) {
  if (!layers || n_layers < 2) fail(TEMCO_ERR_INVALID_ARGUMENT, "need at least an input and one layer");
  if (cfg.batch <= 0 || cfg.height <= 0 || cfg.width <= 0 || cfg.channels <= 0)
    fail(TEMCO_ERR_INVALID_ARGUMENT, "config sizes must be positive");
  if (n_decomps > 0 && !decomps) fail(TEMCO_ERR_INVALID_ARGUMENT, "decomps is NULL");
  if (n_edges > 0 && !edges) fail(TEMCO_ERR_INVALID_ARGUMENT, "skip_edges is NULL");
  (void)bf16;

  std::vector<const temco_decomp*> dec(n_layers, nullptr);
  for (int i = 0; i < n_decomps; ++i) {
    const temco_decomp& d = decomps[i];
    if (d.layer <= 0 || d.layer >= n_layers) fail(TEMCO_ERR_INVALID_GRAPH, "decomp refers to a bad layer");
    if (layers[d.layer].op != TEMCO_OP_CONV2D && layers[d.layer].op != TEMCO_OP_CONV_TRANSPOSE2D)
      fail(TEMCO_ERR_INVALID_GRAPH, "decomp of a non-conv layer");
    if (dec[d.layer]) fail(TEMCO_ERR_INVALID_GRAPH, "two decomps for one layer");
    dec[d.layer] = &d;
  }

  // declared skip edges == computed (dst - src > 1)
  std::set<std::pair<int, int>> want, got;
  for (int i = 0; i < n_layers; ++i) {
    const temco_layer& l = layers[i];
    if (l.n_inputs < 0 || (l.n_inputs > 0 && !l.inputs)) fail(TEMCO_ERR_INVALID_ARGUMENT, "bad inputs array");
    for (int k = 0; k < l.n_inputs; ++k)
      if (l.inputs[k] >= 0 && i - l.inputs[k] > 1) want.insert({l.inputs[k], i});
  }
  for (int i = 0; i < n_edges; ++i) got.insert({edges[i].src, edges[i].dst});
  if (want != got) fail(TEMCO_ERR_INVALID_GRAPH, "skip_edges differ from the graph's dst-src>1 input edges");

  std::vector<int> out_of(n_layers, -1);
  auto push = [&](Node n) {
    n.id = (int)ir.nodes.size();
    if (n.H <= 0 || n.W <= 0 || n.C <= 0) fail(TEMCO_ERR_INVALID_GRAPH, "non-positive inferred shape");
    ir.nodes.push_back(std::move(n));
    return ir.nodes.back().id;
  };

  for (int li = 0; li < n_layers; ++li) {
    const temco_layer& l = layers[li];
    std::vector<int> ins;
    for (int k = 0; k < l.n_inputs; ++k) {
      int s = l.inputs[k];
      if (s < 0 || s >= li) fail(TEMCO_ERR_INVALID_GRAPH, "inputs must refer to earlier layers (SSA order)");
      ins.push_back(out_of[s]);
    }
    auto need = [&](int n) {
      if ((int)ins.size() != n) fail(TEMCO_ERR_INVALID_GRAPH, "wrong number of inputs");
    };
    Node n;
    n.orig = li;
    if (li == 0) {
      if (l.op != TEMCO_OP_INPUT) fail(TEMCO_ERR_INVALID_GRAPH, "layer 0 must be the input");
      n.op = OP_INPUT;
      n.C = cfg.channels; n.H = cfg.height; n.W = cfg.width;
      out_of[li] = push(n);
      continue;
    }
    if (l.op == TEMCO_OP_INPUT) fail(TEMCO_ERR_INVALID_GRAPH, "only layer 0 may be an input");
    switch (l.op) {
      case TEMCO_OP_CONV2D: {
        need(1);
        const Node x = ir.nodes[ins[0]];
        int k = l.kernel, s = l.stride, p = l.pad, g = l.groups <= 0 ? 1 : l.groups;
        if (k <= 0 || s <= 0 || p < 0 || l.out_channels <= 0) fail(TEMCO_ERR_INVALID_GRAPH, "bad conv params");
        if (x.C % g || l.out_channels % g) fail(TEMCO_ERR_INVALID_GRAPH, "groups must divide channels");
        int ho = (x.H + 2 * p - k) / s + 1, wo = (x.W + 2 * p - k) / s + 1;
        if (x.H + 2 * p < k || x.W + 2 * p < k) fail(TEMCO_ERR_INVALID_GRAPH, "conv kernel larger than input");
        // original conv FLOPs: COMPUTE_THRESHOLD (reading R1)
        ir.orig_flops[li] = 2LL * (x.C / g) * l.out_channels * k * k * (int64_t)ho * wo * cfg.batch;
        const temco_decomp* d = dec[li];
        if (!d) {
          if (!l.weight) fail(TEMCO_ERR_INVALID_ARGUMENT, "undecomposed conv needs a weight");
          n.op = OP_CONV; n.kh = n.kw = k; n.sh = n.sw = s; n.ph = n.pw = p; n.groups = g;
          n.C = l.out_channels; n.H = ho; n.W = wo;
          n.w = copy_buf(l.weight, (size_t)l.out_channels * (x.C / g) * k * k);
          n.b = copy_buf(l.bias, l.out_channels);
          n.in = ins;
          out_of[li] = push(n);
          break;
        }
        if (g != 1) fail(TEMCO_ERR_UNSUPPORTED, "decomposed grouped convolutions are not supported");
        if (d->rank_in <= 0 || d->rank_out <= 0) fail(TEMCO_ERR_UNSUPPORTED, "ranks must be positive");
        if (d->kind == TEMCO_DECOMP_TUCKER2) {
          int ri = d->rank_in, ro = d->rank_out;
          if (ri > x.C || ro > l.out_channels) fail(TEMCO_ERR_UNSUPPORTED, "Tucker-2 rank exceeds its mode");
          if (!d->core) fail(TEMCO_ERR_INVALID_ARGUMENT, "Tucker-2 core is NULL");
          if ((ri < x.C && !d->first) || (ro < l.out_channels && !d->last))
            fail(TEMCO_ERR_INVALID_ARGUMENT, "reduced Tucker-2 mode without its factor");
          int cur = ins[0];
          if (d->first) {
            Node f; f.op = OP_CONV; f.role = ROLE_FCONV; f.orig = li; f.in = {cur};
            f.C = ri; f.H = x.H; f.W = x.W;
            f.w = copy_buf(d->first, (size_t)ri * x.C);
            cur = push(f);
          } else if (ri != x.C) {
            fail(TEMCO_ERR_INVALID_GRAPH, "rank_in != C_in requires a first factor");
          }
          Node c; c.op = OP_CONV; c.role = ROLE_CORE; c.orig = li; c.in = {cur};
          c.kh = c.kw = k; c.sh = c.sw = s; c.ph = c.pw = p; c.C = ro; c.H = ho; c.W = wo;
          c.w = copy_buf(d->core, (size_t)ro * ri * k * k);
          if (!d->last) c.b = copy_buf(l.bias, ro);
          cur = push(c);
          if (d->last) {
            Node q; q.op = OP_CONV; q.role = ROLE_LCONV; q.orig = li; q.in = {cur};
            q.C = l.out_channels; q.H = ho; q.W = wo;
            q.w = copy_buf(d->last, (size_t)l.out_channels * ro);
            q.b = copy_buf(l.bias, l.out_channels);
            cur = push(q);
          } else if (ro != l.out_channels) {
            fail(TEMCO_ERR_INVALID_GRAPH, "rank_out != C_out requires a last factor");
          }
          out_of[li] = cur;
        } else if (d->kind == TEMCO_DECOMP_CP) {
          int r = d->rank_in;
          if (d->rank_out != r) fail(TEMCO_ERR_INVALID_ARGUMENT, "CP needs rank_in == rank_out");
          if (!d->first || !d->core || !d->core2 || !d->last) fail(TEMCO_ERR_INVALID_ARGUMENT, "CP factor is NULL");
          Node f; f.op = OP_CONV; f.role = ROLE_FCONV; f.orig = li; f.in = {ins[0]};
          f.C = r; f.H = x.H; f.W = x.W; f.w = copy_buf(d->first, (size_t)r * x.C);
          int fi = push(f);
          int h1 = (x.H + 2 * p - k) / s + 1;
          Node v; v.op = OP_CONV; v.role = ROLE_CORE; v.orig = li; v.in = {fi};
          v.kh = k; v.kw = 1; v.sh = s; v.sw = 1; v.ph = p; v.pw = 0; v.groups = r;
          v.C = r; v.H = h1; v.W = x.W; v.w = copy_buf(d->core, (size_t)r * k);
          int vi = push(v);
          Node h; h.op = OP_CONV; h.role = ROLE_CORE; h.orig = li; h.in = {vi};
          h.kh = 1; h.kw = k; h.sh = 1; h.sw = s; h.ph = 0; h.pw = p; h.groups = r;
          h.C = r; h.H = ho; h.W = wo; h.w = copy_buf(d->core2, (size_t)r * k);
          int hi = push(h);
          Node q; q.op = OP_CONV; q.role = ROLE_LCONV; q.orig = li; q.in = {hi};
          q.C = l.out_channels; q.H = ho; q.W = wo;
          q.w = copy_buf(d->last, (size_t)l.out_channels * r);
          q.b = copy_buf(l.bias, l.out_channels);
          out_of[li] = push(q);
        } else if (d->kind == TEMCO_DECOMP_TT) {
          // Tensor-Train (P:L73 [28]; reading R33): fconv 1x1 (C_in -> r1, omitted when
          // r1 == C_in) -> K x 1 conv (r1 -> r2) -> 1 x K conv (r2 -> r3) -> lconv 1x1 (r3 -> C_out)
          const int r1 = d->rank_in, r2 = d->rank_mid, r3 = d->rank_out;
          if (r2 <= 0) fail(TEMCO_ERR_UNSUPPORTED, "ranks must be positive");
          if (!d->core || !d->core2 || !d->last) fail(TEMCO_ERR_INVALID_ARGUMENT, "TT factor is NULL");
          if (r1 > x.C) fail(TEMCO_ERR_UNSUPPORTED, "TT rank exceeds its mode");
          int cur = ins[0];
          if (d->first) {
            Node f; f.op = OP_CONV; f.role = ROLE_FCONV; f.orig = li; f.in = {cur};
            f.C = r1; f.H = x.H; f.W = x.W; f.w = copy_buf(d->first, (size_t)r1 * x.C);
            cur = push(f);
          } else if (r1 != x.C) {
            fail(TEMCO_ERR_INVALID_GRAPH, "rank_in != C_in requires a first factor");
          }
          const int h1 = (x.H + 2 * p - k) / s + 1;
          Node v; v.op = OP_CONV; v.role = ROLE_CORE; v.orig = li; v.in = {cur};
          v.kh = k; v.kw = 1; v.sh = s; v.sw = 1; v.ph = p; v.pw = 0;
          v.C = r2; v.H = h1; v.W = x.W; v.w = copy_buf(d->core, (size_t)r2 * r1 * k);
          const int vi = push(v);
          Node h; h.op = OP_CONV; h.role = ROLE_CORE; h.orig = li; h.in = {vi};
          h.kh = 1; h.kw = k; h.sh = 1; h.sw = s; h.ph = 0; h.pw = p;
          h.C = r3; h.H = ho; h.W = wo; h.w = copy_buf(d->core2, (size_t)r3 * r2 * k);
          const int hi = push(h);
          Node q; q.op = OP_CONV; q.role = ROLE_LCONV; q.orig = li; q.in = {hi};
          q.C = l.out_channels; q.H = ho; q.W = wo;
          q.w = copy_buf(d->last, (size_t)l.out_channels * r3);
          q.b = copy_buf(l.bias, l.out_channels);
          out_of[li] = push(q);
        } else {
          fail(TEMCO_ERR_INVALID_ARGUMENT, "unknown decomposition kind");
        }
        break;
      }
      case TEMCO_OP_CONV_TRANSPOSE2D: {
        // transposed conv: out[h*s + i - p, w*s + j - p, o] += x[h, w, c] W[c, o, i, j]
        need(1);
        const Node x = ir.nodes[ins[0]];
        const int k = l.kernel, s = l.stride, p = l.pad;
        if (k <= 0 || s <= 0 || p < 0 || l.out_channels <= 0 || (l.groups > 1)) fail(TEMCO_ERR_INVALID_GRAPH, "bad conv_transpose params");
        const int ho = (x.H - 1) * s - 2 * p + k, wo = (x.W - 1) * s - 2 * p + k;
        if (ho <= 0 || wo <= 0) fail(TEMCO_ERR_INVALID_GRAPH, "conv_transpose output is empty");
        // original FLOPs (reading R1): every input pixel meets every k x k tap
        ir.orig_flops[li] = 2LL * x.C * l.out_channels * k * k * (int64_t)x.H * x.W * cfg.batch;
        const temco_decomp* d = dec[li];
        if (!d) {
          if (!l.weight) fail(TEMCO_ERR_INVALID_ARGUMENT, "undecomposed conv_transpose needs a weight");
          n.op = OP_CONVT; n.kh = n.kw = k; n.sh = n.sw = s; n.ph = n.pw = p;
          n.C = l.out_channels; n.H = ho; n.W = wo;
          n.w = copy_buf(l.weight, (size_t)x.C * l.out_channels * k * k);
          n.b = copy_buf(l.bias, l.out_channels);
          n.in = ins;
          out_of[li] = push(n);
          break;
        }
        if (d->kind != TEMCO_DECOMP_TUCKER2) fail(TEMCO_ERR_UNSUPPORTED, "conv_transpose: Tucker-2 decomposition only");
        const int ri = d->rank_in, ro = d->rank_out;
        if (ri <= 0 || ro <= 0 || ri > x.C || ro > l.out_channels) fail(TEMCO_ERR_UNSUPPORTED, "bad conv_transpose ranks");
        if (!d->core || (ri < x.C && !d->first) || (ro < l.out_channels && !d->last))
          fail(TEMCO_ERR_INVALID_ARGUMENT, "conv_transpose factor is NULL");
        int cur = ins[0];
        if (d->first) {
          Node f; f.op = OP_CONV; f.role = ROLE_FCONV; f.orig = li; f.in = {cur};
          f.C = ri; f.H = x.H; f.W = x.W;
          f.w = copy_buf(d->first, (size_t)ri * x.C);
          cur = push(f);
        } else if (ri != x.C) {
          fail(TEMCO_ERR_INVALID_GRAPH, "rank_in != C_in requires a first factor");
        }
        Node c; c.op = OP_CONVT; c.role = ROLE_CORE; c.orig = li; c.in = {cur};
        c.kh = c.kw = k; c.sh = c.sw = s; c.ph = c.pw = p; c.C = ro; c.H = ho; c.W = wo;
        c.w = copy_buf(d->core, (size_t)ri * ro * k * k);
        if (!d->last) c.b = copy_buf(l.bias, ro);
        cur = push(c);
        if (d->last) {
          Node q; q.op = OP_CONV; q.role = ROLE_LCONV; q.orig = li; q.in = {cur};
          q.C = l.out_channels; q.H = ho; q.W = wo;
          q.w = copy_buf(d->last, (size_t)l.out_channels * ro);
          q.b = copy_buf(l.bias, l.out_channels);
          cur = push(q);
        } else if (ro != l.out_channels) {
          fail(TEMCO_ERR_INVALID_GRAPH, "rank_out != C_out requires a last factor");
        }
        out_of[li] = cur;
        break;
      }
      case TEMCO_OP_BATCHNORM: {
        need(1);
        const Node& x = ir.nodes[ins[0]];
        if (!l.bn_gamma || !l.bn_beta || !l.bn_mean || !l.bn_var) fail(TEMCO_ERR_INVALID_ARGUMENT, "BN params NULL");
        n.op = OP_BN; n.C = x.C; n.H = x.H; n.W = x.W; n.in = ins; n.eps = l.bn_eps;
        n.bn_g = copy_buf(l.bn_gamma, x.C); n.bn_b = copy_buf(l.bn_beta, x.C);
        n.bn_m = copy_buf(l.bn_mean, x.C); n.bn_v = copy_buf(l.bn_var, x.C);
        out_of[li] = push(n);
        break;
      }
      case TEMCO_OP_RELU:
      case TEMCO_OP_SILU: {
        need(1);
        const Node& x = ir.nodes[ins[0]];
        n.op = l.op == TEMCO_OP_RELU ? OP_RELU : OP_SILU; n.C = x.C; n.H = x.H; n.W = x.W; n.in = ins;
        out_of[li] = push(n);
        break;
      }
      case TEMCO_OP_ADD: {
        if (ins.size() < 2) fail(TEMCO_ERR_INVALID_GRAPH, "add needs >= 2 inputs");
        const Node& x = ir.nodes[ins[0]];
        for (int s : ins) {
          const Node& y = ir.nodes[s];
          if (y.C != x.C || y.H != x.H || y.W != x.W) fail(TEMCO_ERR_INVALID_GRAPH, "add shape mismatch");
        }
        n.op = OP_ADD; n.C = x.C; n.H = x.H; n.W = x.W; n.in = ins;
        out_of[li] = push(n);
        break;
      }
      case TEMCO_OP_CONCAT: {
        if (ins.empty()) fail(TEMCO_ERR_INVALID_GRAPH, "concat needs inputs");
        const Node& x = ir.nodes[ins[0]];
        int c = 0;
        for (int s : ins) {
          const Node& y = ir.nodes[s];
          if (y.H != x.H || y.W != x.W) fail(TEMCO_ERR_INVALID_GRAPH, "concat spatial mismatch");
          c += y.C;
        }
        n.op = OP_CONCAT; n.C = c; n.H = x.H; n.W = x.W; n.in = ins;
        out_of[li] = push(n);
        break;
      }
      case TEMCO_OP_MAXPOOL:
      case TEMCO_OP_AVGPOOL: {
        need(1);
        const Node& x = ir.nodes[ins[0]];
        int k = l.kernel, s = l.stride, p = l.op == TEMCO_OP_MAXPOOL ? l.pad : 0;
        if (k <= 0 || s <= 0 || p < 0 || 2 * p > k) fail(TEMCO_ERR_INVALID_GRAPH, "bad pool params");
        n.op = l.op == TEMCO_OP_MAXPOOL ? OP_MAXPOOL : OP_AVGPOOL;
        n.kh = n.kw = k; n.sh = n.sw = s; n.ph = n.pw = p;
        n.C = x.C; n.H = (x.H + 2 * p - k) / s + 1; n.W = (x.W + 2 * p - k) / s + 1; n.in = ins;
        if (x.H + 2 * p < k || x.W + 2 * p < k) fail(TEMCO_ERR_INVALID_GRAPH, "pool window larger than input");
        out_of[li] = push(n);
        break;
      }
      case TEMCO_OP_GLOBAL_AVGPOOL: {
        need(1);
        const Node& x = ir.nodes[ins[0]];
        n.op = OP_GAP; n.C = x.C; n.H = 1; n.W = 1; n.in = ins;
        out_of[li] = push(n);
        break;
      }
      case TEMCO_OP_LINEAR: {
        need(1);
        const Node& x = ir.nodes[ins[0]];
        if (!l.weight || l.out_channels <= 0) fail(TEMCO_ERR_INVALID_ARGUMENT, "linear needs weight / out_channels");
        n.op = OP_LINEAR; n.C = l.out_channels; n.H = 1; n.W = 1; n.in = ins;
        n.w = copy_buf(l.weight, (size_t)l.out_channels * x.C * x.H * x.W);
        n.b = copy_buf(l.bias, l.out_channels);
        out_of[li] = push(n);
        break;
      }
      default:
        fail(TEMCO_ERR_UNSUPPORTED, "unsupported operator");
    }
  }
  ir.nL = (int)ir.nodes.size();
  ir.output = out_of[n_layers - 1];
  ir.input = 0;
}

// ---------------------------------------------------------------------------
// peak accounting over a list of steps (Eq. (3)/(4), reading R14)
// ---------------------------------------------------------------------------
int64_t peak_of(const IR& ir, const std::vector<Step>& steps, std::vector<int64_t>& live) {
  const int T = (int)steps.size();
  std::map<int, int> def, last;
  for (int t = 0; t < T; ++t) {
    std::vector<int> outs = {steps[t].out};
    outs.insert(outs.end(), steps[t].extra.begin(), steps[t].extra.end());
    for (int o : outs) {
      def[o] = t;
      if (!last.count(o)) last[o] = t;
    }
    for (int x : steps[t].in) last[x] = t;
  }
  last[ir.output] = T - 1;
  // difference array over [def, last]
  std::vector<int64_t> delta(T + 1, 0);
  for (auto& kv : def) {
    int x = kv.first;
    delta[kv.second] += ir.size(x);
    delta[last[x] + 1] -= ir.size(x);
  }
  live.assign(T, 0);
  int64_t cur = 0, best = 0;
  for (int t = 0; t < T; ++t) {
    cur += delta[t];
    live[t] = cur;
    best = std::max(best, cur);
  }
  return best;
}

// ---------------------------------------------------------------------------
// Alg. 2
// ---------------------------------------------------------------------------
struct Res {
  bool ok = false;
  std::vector<int> list;
  int64_t size = 0, peak = 0;
};

int64_t peak_alg2(const std::vector<Res>& l, int64_t size_v) {   // Peak(l, v)
  int64_t peak = 0, resided = 0;
  for (const Res& e : l) {
    peak = std::max(resided + e.peak, peak);
    resided += e.size;
  }
  return std::max(resided + size_v, peak);
}

Res find_reduced(const IR& ir, int v) {   // FindReduced(v, G) on PDG(L)
  const Node& n = ir.nodes[v];
  Res r;
  if (is_lconv(n)) {
    r.ok = true;
    r.list = {v};
    r.size = ir.size(v);
    r.peak = ir.size(v) + ir.size(n.in[0]);
    return r;
  }
  if (!recurse_op(n.op)) return r;   // input / non-lconv conv / linear / GAP: fail (R6)
  std::vector<Res> preds;
  for (int p : n.in) {
    Res q = find_reduced(ir, p);
    if (!q.ok) return r;
    preds.push_back(std::move(q));
  }
  // ORDER(Compare): Compare(a,b) <=> a.size - a.peak < b.size - b.peak; stable (R8)
  std::stable_sort(preds.begin(), preds.end(),
                   [](const Res& a, const Res& b) { return a.size + b.peak < b.size + a.peak; });
  for (const Res& e : preds)
    for (int x : e.list)
      if (std::find(r.list.begin(), r.list.end(), x) == r.list.end()) r.list.push_back(x);
  r.list.push_back(v);
  r.ok = true;
  r.size = ir.size(v);
  r.peak = peak_alg2(preds, r.size);
  return r;
}

}  // namespace

int64_t node_flops(const IR& ir, int id) {   // reading R1
  const Node& v = ir.nodes[id];
  const int64_t N = ir.batch;
  const int64_t numel = N * v.C * v.H * v.W;
  switch (v.op) {
    case OP_CONV: {
      const Node& x = ir.nodes[v.in[0]];
      return 2LL * (x.C / v.groups) * v.C * v.kh * v.kw * (int64_t)v.H * v.W * N;
    }
    case OP_CONVT: {   // per input pixel: C_in x C_out x k x k MACs
      const Node& x = ir.nodes[v.in[0]];
      return 2LL * x.C * v.C * v.kh * v.kw * (int64_t)x.H * x.W * N;
    }
    case OP_BN: return 2 * numel;
    case OP_RELU: return numel;
    case OP_SILU: return 4 * numel;
    case OP_ADD: return (int64_t)(v.in.size() - 1) * numel;
    case OP_MAXPOOL:
    case OP_AVGPOOL: return (int64_t)v.kh * v.kw * numel;
    case OP_GAP: {
      const Node& x = ir.nodes[v.in[0]];
      return N * x.C * x.H * x.W;
    }
    case OP_LINEAR: {
      const Node& x = ir.nodes[v.in[0]];
      return 2LL * x.C * x.H * x.W * v.C * N;
    }
    default: return 0;
  }
}

namespace {

// Overhead(n, l): Alg. 1 lines 1-9, P:L188 / P:L219, reading R1
bool overhead(const IR& ir, const Res& l, int64_t m, int policy) {
  if (policy == 1) return true;
  if (policy == 2) return false;
  int64_t c = 0, thr = 0;
  std::vector<int> origs;
  for (int x : l.list) {
    c += node_flops(ir, x);
    const Node& v = ir.nodes[x];
    if (is_lconv(v) && std::find(origs.begin(), origs.end(), v.orig) == origs.end()) {
      origs.push_back(v.orig);
      thr += ir.orig_flops.at(v.orig);
    }
  }
  return c <= thr && l.peak <= m;
}

void skip_opt(IR& ir, const BuildOptions& opt) {
  const int nL = ir.nL;
  // liveness on L (Alg. 1 lines 10-16): ids are positions in L
  std::vector<int> begin(nL), end(nL);
  std::vector<std::vector<int>> succ(nL);
  for (int i = 0; i < nL; ++i) {
    begin[i] = i;
    end[i] = i;
  }
  for (int i = 0; i < nL; ++i)
    for (int p : ir.nodes[i].in) {
      end[p] = i;
      if (std::find(succ[p].begin(), succ[p].end(), i) == succ[p].end()) succ[p].push_back(i);
    }
  end[ir.output] = nL - 1;

  for (int n = 0; n < nL; ++n) {                          // line 17
    if (end[n] - begin[n] <= opt.distance_threshold) continue;   // lines 18-19
    Res l = find_reduced(ir, n);                          // line 20
    if (!l.ok) {
      ir.decisions.push_back({n, 1, {}});
      continue;
    }
    if (!overhead(ir, l, ir.peak_unfused, opt.overhead_policy)) {   // line 21
      ir.decisions.push_back({n, 2, {}});
      continue;
    }
    ir.decisions.push_back({n, 0, l.list});
    for (int s : succ[n]) {                               // line 22
      if (s - n <= opt.distance_threshold) continue;      // near use keeps the original (R4)
      std::map<int, int> copy;                            // COPY(l.list), fresh ids (R5)
      std::vector<int> fresh;
      for (int x : l.list) {
        Node c = ir.nodes[x];
        c.id = (int)ir.nodes.size();
        c.copy_of = x;
        for (int& i : c.in) {
          auto it = copy.find(i);
          if (it != copy.end()) i = it->second;
        }
        copy[x] = c.id;
        fresh.push_back(c.id);
        ir.oin.push_back(c.in);
        ir.nodes.push_back(std::move(c));
      }
      auto at = std::find(ir.O.begin(), ir.O.end(), s);   // InsertBefore(O, s, …), line 23
      ir.O.insert(at, fresh.begin(), fresh.end());
      for (int& i : ir.oin[s])                            // replace the skip
        if (i == n) i = copy[n];
    }
  }
}

void dce(IR& ir) {   // reading R11
  while (true) {
    std::set<int> used;
    for (int x : ir.O)
      for (int p : ir.oin[x]) used.insert(p);
    std::vector<int> keep;
    for (int x : ir.O)
      if (used.count(x) || x == ir.input || x == ir.output) keep.push_back(x);
    if (keep.size() == ir.O.size()) return;
    ir.O.swap(keep);
  }
}

// reading R35 (oracle: fold_1x1_cores): an unstrided, unpadded, ungrouped, bias-free 1x1 core
// whose input is an fconv read by nothing else folds into that fconv (two linear 1x1 maps):
// the core's node becomes the fconv with weight G F, the fconv leaves O
void fold_1x1_cores(IR& ir) {
  std::map<int, std::vector<int>> cons;
  for (int x : ir.O) {
    std::vector<int> seen;
    for (int p : ir.oin[x])
      if (std::find(seen.begin(), seen.end(), p) == seen.end()) {
        seen.push_back(p);
        cons[p].push_back(x);
      }
  }
  std::set<int> drop;
  for (int x : ir.O) {
    Node& c = ir.nodes[x];
    if (!(c.op == OP_CONV && c.role == ROLE_CORE && c.kh == 1 && c.kw == 1 && c.sh == 1 && c.sw == 1 && c.ph == 0 &&
          c.pw == 0 && c.groups == 1 && !c.b && ir.oin[x].size() == 1))
      continue;
    const int fi = ir.oin[x][0];
    const Node& f = ir.nodes[fi];
    if (fi == ir.input || f.op != OP_CONV || f.role != ROLE_FCONV || f.kh != 1 || f.kw != 1 || f.b) continue;
    if (cons[fi].size() != 1 || cons[fi][0] != x) continue;
    const int R_out = c.C, R_in = f.C, Cin = ir.nodes[ir.oin[fi][0]].C;
    auto w = std::make_shared<std::vector<float>>((size_t)R_out * Cin, 0.f);
    for (int o = 0; o < R_out; ++o)
      for (int k = 0; k < R_in; ++k) {
        const double g = (*c.w)[(size_t)o * R_in + k];
        for (int i = 0; i < Cin; ++i) (*w)[(size_t)o * Cin + i] += (float)(g * (*f.w)[(size_t)k * Cin + i]);
      }
    c.role = ROLE_FCONV;
    c.w = w;
    c.in = f.in;
    ir.oin[x] = ir.oin[fi];
    drop.insert(fi);
  }
  std::vector<int> O;
  for (int x : ir.O)
    if (!drop.count(x)) O.push_back(x);
  ir.O = O;
}

// reading R36 (oracle: pool_before_restore): avgpool(lconv(r)) = lconv(avgpool(r)); each pooled
// restore copy becomes a plain restore of ONE shared pooled reduced tensor placed right after r
void pool_before_restore(IR& ir) {
  std::map<int, std::vector<int>> cons;
  for (int x : ir.O) {
    std::vector<int> seen;
    for (int p : ir.oin[x])
      if (std::find(seen.begin(), seen.end(), p) == seen.end()) {
        seen.push_back(p);
        cons[p].push_back(x);
      }
  }
  std::map<std::tuple<int, int, int, int, int>, int> shared;
  std::map<int, std::vector<int>> placed;   // r -> pooled nodes to insert after it
  std::set<int> drop;
  for (int x : ir.O) {
    const Node a = ir.nodes[x];
    if (a.op != OP_AVGPOOL || ir.oin[x].size() != 1) continue;
    const int li = ir.oin[x][0];
    const Node l = ir.nodes[li];
    if (!(l.op == OP_CONV && l.role == ROLE_LCONV && l.kh == 1 && l.kw == 1 && l.sh == 1 && l.sw == 1 &&
          l.groups == 1 && cons[li].size() == 1 && cons[li][0] == x))
      continue;
    const int ri = ir.oin[li][0];
    const Node& r = ir.nodes[ri];
    const auto key = std::make_tuple(ri, a.kh, a.kw, a.sh, a.sw);
    auto it = shared.find(key);
    int pid;
    if (it == shared.end()) {
      Node p;
      p.op = OP_AVGPOOL; p.orig = a.orig; p.in = {ri};
      p.kh = a.kh; p.kw = a.kw; p.sh = a.sh; p.sw = a.sw; p.ph = a.ph; p.pw = a.pw;
      p.C = r.C; p.H = a.H; p.W = a.W;
      pid = (int)ir.nodes.size();
      p.id = pid;
      ir.oin.push_back({ri});
      ir.nodes.push_back(std::move(p));
      shared[key] = pid;
      placed[ri].push_back(pid);
    } else {
      pid = it->second;
    }
    Node q = l;          // the pooled node becomes the restore of the pooled reduced tensor
    q.id = x;
    q.in = {pid};
    q.H = a.H;
    q.W = a.W;
    q.copy_of = l.copy_of;
    ir.nodes[x] = q;
    ir.oin[x] = {pid};
    drop.insert(li);
  }
  if (shared.empty()) return;
  std::vector<int> O;
  for (int x : ir.O) {
    if (drop.count(x)) continue;
    O.push_back(x);
    auto pl = placed.find(x);
    if (pl != placed.end()) O.insert(O.end(), pl->second.begin(), pl->second.end());
  }
  ir.O = O;
}

void group_and_schedule(IR& ir, bool fusion, bool extensions) {
  std::map<int, int> pos;
  for (size_t i = 0; i < ir.O.size(); ++i) pos[ir.O[i]] = (int)i;
  std::map<int, std::vector<int>> cons;
  for (int x : ir.O) {
    std::vector<int> seen;
    for (int p : ir.oin[x])
      if (std::find(seen.begin(), seen.end(), p) == seen.end()) {
        seen.push_back(p);
        cons[p].push_back(x);
      }
  }
  std::set<int> grouped;
  if (fusion) {
    for (int r : ir.O) {
      const Node& v = ir.nodes[r];
      bool root = false;
      if (v.role == ROLE_FCONV && absorbable(ir.nodes[ir.oin[r][0]])) root = true;
      else if (v.op == OP_GAP && absorbable(ir.nodes[ir.oin[r][0]])) root = true;
      else if (absorbable(v)) {
        if (r == ir.output) root = true;
        for (int c : cons[r])
          if (ir.nodes[c].op == OP_LINEAR) root = true;
      }
      if (!root || grouped.count(r)) continue;
      std::set<int> mem = {r};
      bool changed = true;
      while (changed) {
        changed = false;
        std::vector<int> cur(mem.begin(), mem.end());
        for (int x : cur) {
          if (is_lconv(ir.nodes[x])) continue;            // stop at lconv: its input is a group input
          for (int p : ir.oin[x]) {
            if (mem.count(p) || grouped.count(p) || p == ir.input) continue;
            if (!absorbable(ir.nodes[p])) continue;
            bool all_in = true;
            for (int c : cons[p])
              if (!mem.count(c)) all_in = false;
            if (all_in) {
              mem.insert(p);
              changed = true;
            }
          }
        }
      }
      bool has_lconv = false;
      for (int x : mem) has_lconv |= is_lconv(ir.nodes[x]);
      if (!has_lconv) continue;
      std::vector<int> ms(mem.begin(), mem.end());
      std::sort(ms.begin(), ms.end(), [&](int a, int b) { return pos[a] < pos[b]; });
      ir.groups[r] = ms;
      grouped.insert(mem.begin(), mem.end());
    }
  }
  if (fusion && extensions) {
    // reading R34: the K x 1 and 1 x K depthwise cores of one CP decomposition
    // form one step when the K x 1 output has no other consumer (oracle: pair_cp_cores)
    for (int x : ir.O) {
      const Node& h = ir.nodes[x];
      if (h.op != OP_CONV || ir.oin[x].size() != 1 || grouped.count(x)) continue;
      const int vi = ir.oin[x][0];
      const Node& v = ir.nodes[vi];
      if (grouped.count(vi) || cons[vi].size() != 1 || cons[vi][0] != x) continue;
      const bool pair = v.op == OP_CONV && v.role == ROLE_CORE && h.role == ROLE_CORE && v.orig == h.orig &&
                        v.groups == v.C && h.groups == h.C && v.C == h.C && v.kw == 1 && v.kh > 1 && h.kh == 1 &&
                        h.kw > 1;
      if (!pair) continue;
      ir.groups[x] = {vi, x};
      grouped.insert(vi);
      grouped.insert(x);
    }
  }
  std::map<int, int> member_of;
  for (auto& kv : ir.groups)
    for (int x : kv.second) member_of[x] = kv.first;
  ir.steps.clear();
  for (int x : ir.O) {
    auto it = member_of.find(x);
    Step s;
    if (it != member_of.end()) {
      if (it->second != x) continue;
      s.group = true;
      s.out = x;
      s.members = ir.groups[x];
      std::set<int> ms(s.members.begin(), s.members.end());
      for (int y : s.members)
        for (int p : ir.oin[y])
          if (!ms.count(p) && std::find(s.in.begin(), s.in.end(), p) == s.in.end()) s.in.push_back(p);
    } else {
      s.out = x;
      s.members = {x};
      for (int p : ir.oin[x])
        if (std::find(s.in.begin(), s.in.end(), p) == s.in.end()) s.in.push_back(p);
    }
    ir.steps.push_back(std::move(s));
  }
}

// reading R37 (oracle: restore_key / merge_fconvs): merged-fconv CSE.  A member's identity is the
// node of L it was COPY'd from (Alg. 1 line 23; the root of a copy chain) with its attributes and
// the identities of its inputs; a tensor from outside the group is identified by its id.
int copy_root(const IR& ir, int x) {
  const int c = ir.nodes[x].copy_of;
  if (c < 0) return x;
  int b = c;
  while (ir.nodes[b].copy_of >= 0) b = ir.nodes[b].copy_of;
  return b;
}

void restore_key(const IR& ir, const std::set<int>& mem, int x, std::vector<int64_t>& k) {
  if (!mem.count(x)) {
    k.push_back(-1);
    k.push_back(x);
    return;
  }
  const Node& v = ir.nodes[x];
  const int64_t a[] = {-2, copy_root(ir, x), v.op, v.role, v.kh, v.kw, v.sh, v.sw, v.ph, v.pw, v.groups, v.C, v.H,
                       v.W, (int64_t)ir.oin[x].size()};
  k.insert(k.end(), a, a + sizeof(a) / sizeof(a[0]));
  for (int i : ir.oin[x]) restore_key(ir, mem, i, k);
  k.push_back(-3);
}

// taking the fused groups in S order, a later group whose fconv root reads a tensor with the same
// key as an earlier group's root runs its reduce in the earlier group's step (its other members
// leave O); kept iff the fused peak does not grow (policy 1: iff it stays <= the unfused peak m)
void merge_fconvs(IR& ir, int policy) {
  std::vector<int64_t> scratch;
  int64_t cur = peak_of(ir, ir.steps, scratch);
  auto fconv_group = [&](const Step& s) { return s.group && ir.nodes[s.out].role == ROLE_FCONV; };
  auto key_of = [&](const Step& s) {
    std::vector<int64_t> k;
    restore_key(ir, std::set<int>(s.members.begin(), s.members.end()), ir.oin[s.out][0], k);
    return k;
  };
  for (size_t i = 0; i < ir.steps.size(); ++i) {
    if (!fconv_group(ir.steps[i])) continue;
    const int ta = ir.oin[ir.steps[i].out][0];
    const std::vector<int64_t> ka = key_of(ir.steps[i]);
    size_t j = i + 1;
    while (j < ir.steps.size()) {
      const Step b = ir.steps[j];
      if (!fconv_group(b) || key_of(b) != ka) {
        ++j;
        continue;
      }
      Step merged = ir.steps[i];
      merged.members.push_back(b.out);
      merged.extra.push_back(b.out);
      std::vector<Step> trial = ir.steps;
      trial[i] = merged;
      trial.erase(trial.begin() + (long)j);
      const int64_t np = peak_of(ir, trial, scratch);
      if (np > (policy == 1 ? ir.peak_unfused : cur)) {
        ++j;
        continue;
      }
      cur = np;
      ir.steps.swap(trial);
      ir.oin[b.out] = {ta};   // b's reduce reads a's restored tensor
      std::set<int> dropped(b.members.begin(), b.members.end());
      std::vector<int> O;
      for (int x : ir.O)
        if (!dropped.count(x)) O.push_back(x);
      auto at = std::find(O.begin(), O.end(), merged.out);
      O.insert(at + (long)merged.extra.size(), b.out);   // right after a's outputs
      ir.O.swap(O);
      ir.groups[merged.out] = merged.members;
      ir.groups.erase(b.out);
    }
  }
}

// reading R38 (oracle: reschedule): the order of S with the least peak (O10), exactly, by dynamic
// programming over the sets of executed steps; among the optimal orders the lexicographically first
// (at every point the earliest step of S whose choice keeps the optimum reachable).  More than
// kMaxStates reachable sets: S is kept.
constexpr size_t kRescheduleMaxStates = 100000;

struct Rescheduler {
  const IR& ir;
  int n = 0, words = 0;
  std::vector<std::vector<int>> outs, deps;          // per step
  std::map<int, std::vector<int>> readers;           // tensor -> reading steps
  std::vector<int64_t> osz;
  std::map<std::vector<uint64_t>, int64_t> memo;
  struct TooMany {};

  static bool has(const std::vector<uint64_t>& X, int v) { return (X[v >> 6] >> (v & 63)) & 1u; }
  static std::vector<uint64_t> with(std::vector<uint64_t> X, int v) {
    X[v >> 6] |= 1ull << (v & 63);
    return X;
  }
  int count(const std::vector<uint64_t>& X) const {
    int c = 0;
    for (uint64_t w : X) c += __builtin_popcountll(w);
    return c;
  }
  bool ready(const std::vector<uint64_t>& X, int v) const {
    if (has(X, v)) return false;
    for (int d : deps[v])
      if (!has(X, d)) return false;
    return true;
  }
  int64_t live(const std::vector<uint64_t>& X) const {
    int64_t tot = 0;
    for (int i = 0; i < n; ++i) {
      if (!has(X, i)) continue;
      for (int o : outs[i]) {
        bool keep = o == ir.output;
        auto it = readers.find(o);
        if (!keep && it != readers.end())
          for (int r : it->second)
            if (!has(X, r)) keep = true;
        if (keep) tot += ir.size(o);
      }
    }
    return tot;
  }
  int64_t best(const std::vector<uint64_t>& X) {
    if (count(X) == n) return 0;
    auto it = memo.find(X);
    if (it != memo.end()) return it->second;
    if (memo.size() >= kRescheduleMaxStates) throw TooMany{};
    const int64_t L = live(X);
    int64_t b = -1;
    for (int v = 0; v < n; ++v) {
      if (!ready(X, v)) continue;
      const int64_t r = std::max(L + osz[v], best(with(X, v)));
      if (b < 0 || r < b) b = r;
    }
    memo[X] = b;
    return b;
  }
};

void reschedule(IR& ir) {
  Rescheduler R{ir};
  const auto& S = ir.steps;
  R.n = (int)S.size();
  R.words = (R.n + 63) / 64;
  std::map<int, int> prod;
  R.outs.resize(R.n);
  R.deps.resize(R.n);
  R.osz.assign(R.n, 0);
  for (int i = 0; i < R.n; ++i) {
    R.outs[i] = {S[i].out};
    R.outs[i].insert(R.outs[i].end(), S[i].extra.begin(), S[i].extra.end());
    for (int o : R.outs[i]) {
      prod[o] = i;
      R.osz[i] += ir.size(o);
    }
  }
  for (int i = 0; i < R.n; ++i)
    for (int x : S[i].in) {
      R.deps[i].push_back(prod.at(x));
      auto& rd = R.readers[x];
      if (std::find(rd.begin(), rd.end(), i) == rd.end()) rd.push_back(i);
    }
  std::vector<uint64_t> X(R.words, 0);
  X = Rescheduler::with(X, 0);
  int64_t opt;
  try {
    opt = std::max(R.osz[0], R.best(X));
  } catch (const Rescheduler::TooMany&) {
    return;
  }
  std::vector<Step> order = {S[0]};
  for (int k = 1; k < R.n; ++k) {
    const int64_t L = R.live(X);
    int pick = -1;
    for (int v = 0; v < R.n && pick < 0; ++v)
      if (R.ready(X, v) && std::max(L + R.osz[v], R.best(Rescheduler::with(X, v))) <= opt) pick = v;
    if (pick < 0) throw std::runtime_error("reschedule: no step keeps the optimum");
    order.push_back(S[pick]);
    X = Rescheduler::with(X, pick);
  }
  ir.steps.swap(order);
}

}  // namespace

temco_status build_ir(const temco_layer* layers, int n_layers, const temco_decomp* decomps, int n_decomps,
                      const temco_edge* edges, int n_edges, const temco_config& cfg, const BuildOptions& opt,
                      IR& ir, std::string& err) {
  try {
    ir = IR();
    ir.batch = cfg.batch;
    ir.elem = opt.bf16 ? 2 : 4;
    expand(layers, n_layers, decomps, n_decomps, edges, n_edges, cfg, opt.bf16, ir);
    // unfused baseline L: every node a step
    for (int i = 0; i < ir.nL; ++i) {
      Step s;
      s.out = i;
      s.members = {i};
      for (int p : ir.nodes[i].in)
        if (std::find(s.in.begin(), s.in.end(), p) == s.in.end()) s.in.push_back(p);
      ir.unfused_steps.push_back(s);
    }
    ir.peak_unfused = peak_of(ir, ir.unfused_steps, ir.live_unfused);   // m
    ir.O.resize(ir.nL);
    std::iota(ir.O.begin(), ir.O.end(), 0);
    ir.oin.resize(ir.nL);
    for (int i = 0; i < ir.nL; ++i) ir.oin[i] = ir.nodes[i].in;
    if (opt.skip_opt) {
      skip_opt(ir, opt);
      dce(ir);
    }
    if (opt.fusion && opt.extensions) {
      fold_1x1_cores(ir);
      pool_before_restore(ir);
    }
    group_and_schedule(ir, opt.fusion, opt.extensions);
    if (opt.fusion && opt.extensions && opt.cse) merge_fconvs(ir, opt.cse_policy);
    if (opt.fusion && opt.extensions && opt.reorder) reschedule(ir);
    ir.peak_fused = peak_of(ir, ir.steps, ir.live_fused);
    return TEMCO_OK;
  } catch (const Fail& f) {
    err = f.msg;
    return f.st;
  } catch (const std::bad_alloc&) {
    err = "host allocation failed";
    return TEMCO_ERR_OUT_OF_MEMORY;
  } catch (const std::exception& e) {
    err = e.what();
    return TEMCO_ERR_INVALID_GRAPH;
  }
}

}  // namespace temco
