// C ABI (include/temco.h): plan creation (planner + lowering + arena +
// uploads), the stream-ordered executor and the host-side queries.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstring>
#include <map>
#include <set>
#include <sstream>
#include <string>
#include <vector>

#include "kernels.h"
#include "planner.h"
#include "conv_tc.h"
#include "mma_chain.h"
#include "tc.h"
#include "tc_wide.h"
#include "pair.h"
#include "gemm.h"
#include "tile.h"


using namespace temco;

namespace {

thread_local std::string g_last_error;

temco_status set_err(temco_status s, const std::string& m) {
  g_last_error = m;
  return s;
}

#define CUDA_TRY(expr)                                                                          \
  do {                                                                                          \
    cudaError_t e_ = (expr);                                                                    \
    if (e_ != cudaSuccess) return set_err(TEMCO_ERR_CUDA, std::string(#expr ": ") + cudaGetErrorString(e_)); \
  } while (0)

enum StepKind { K_NONE, K_CONVT, K_CONV, K_EW, K_LINEAR, K_GROUP_SIMT, K_GROUP_TC, K_CONV_TC, K_GROUP_MMA, K_GROUP_TCW, K_CONV_RK, K_GROUP_CAT, K_GROUP_PAIR, K_GEMM, K_DWPAIR, K_CONV_TILE,
                K_MULTI /* a merged group replayed once per output: the launches of sub_exec[sub] */ };

struct StepExec {
  int kind = K_NONE;
  ConvDesc conv{};
  EwDesc ew{};
  LinearDesc lin{};
  GroupDesc grp{};
  TcChainDesc tc{};
  wide::TcChainDesc tcw{};
  pair::PairDesc pr{};
  GemmDesc gm{};
  ConvTcDesc ctc{};
  MmaChainDesc mma{};
  RankConvDesc rk{};
  TileConvDesc tile{};
  CatDesc cat{};
  DwPairDesc dwp{};
  std::string kernel;
  int64_t flops = 0, io_bytes = 0;
  int launches = 0;
  bool stem = false;   // K_CONV on the tensor-core small-Cin kernel (kernels_stem.cu)
  std::vector<int> sub;   // K_MULTI: indices into temco_plan_s::sub_exec
};

}  // namespace

struct temco_plan_s {
  IR ir;
  temco_config cfg{};
  bool bf16 = false;
  int flags = 0;
  int device = -1;
  bool has_device = false;

  std::vector<StepExec> exec;
  std::vector<StepExec> sub_exec;  // launches of merged groups replayed per output (K_MULTI)
  std::map<int, Loc> loc;
  std::vector<float> params_h;
  std::vector<GNode> gnodes_h;
  std::vector<int32_t> gchild_h;
  std::vector<uint16_t> tcw_h;     // bf16 weight pool of the tcgen05 kernels
  float* params_d = nullptr;
  GNode* gnodes_d = nullptr;
  int32_t* gchild_d = nullptr;
  uint16_t* tcw_d = nullptr;
  char* arena_d = nullptr;
  float* lin_ws_d = nullptr;       // fp32 split-K partials of the tcgen05 GEMM steps
  int64_t lin_ws_elems = 0;
  int64_t arena_bytes = 0;
  int64_t in_bytes = 0, out_bytes = 0;
  void* host_in_d = nullptr;
  void* host_out_d = nullptr;
  // temco_run_host_async: double-buffered staging, copy stream, per-buffer events
  void* async_in_d[2] = {nullptr, nullptr};
  void* async_out_d[2] = {nullptr, nullptr};
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t ev_in_ready[2] = {nullptr, nullptr}, ev_buf_free[2] = {nullptr, nullptr};
  int async_flip = 0;
  int max_expr_depth = 0;          // deepest fused-group expression (SIMT interpreter recursion)
  int64_t out_dims[4] = {0, 0, 0, 0};
  int out_ndim = 0;
  // CUDA graph cache (TEMCO_FLAG_CUDA_GRAPH): one executable graph per (input, output, stream);
  // two entries so temco_run_host_async's alternating staging buffers each keep their graph
  struct GraphEntry {
    cudaGraphExec_t exec = nullptr;
    const void* in = nullptr;
    void* out = nullptr;
    cudaStream_t stream = nullptr;
    uint64_t used = 0;
  } graphs[2];
  uint64_t graph_clock = 0;
  std::string json;
};

namespace {

int64_t push_params(temco_plan_s* P, const std::vector<float>& v) {
  int64_t off = (int64_t)P->params_h.size();
  // keep 16-byte alignment of every parameter block
  P->params_h.insert(P->params_h.end(), v.begin(), v.end());
  while (P->params_h.size() % 4) P->params_h.push_back(0.f);
  return off;
}

int64_t push_params(temco_plan_s* P, const Buf& b) {
  if (!b) return -1;
  return push_params(P, *b);
}

void bn_scale_shift(const Node& n, std::vector<float>& scale, std::vector<float>& shift) {
  scale.resize(n.C);
  shift.resize(n.C);
  for (int c = 0; c < n.C; ++c) {
    double s = (double)(*n.bn_g)[c] / std::sqrt((double)(*n.bn_v)[c] + (double)n.eps);
    scale[c] = (float)s;
    shift[c] = (float)((double)(*n.bn_b)[c] - (double)(*n.bn_m)[c] * s);
  }
}

// conv weight OIHW -> [K][kh][kw][C/groups]
std::vector<float> repack_conv(const Node& n, int cin) {
  const int cg = cin / n.groups;
  std::vector<float> w((size_t)n.C * n.kh * n.kw * cg);
  const std::vector<float>& s = *n.w;
  for (int k = 0; k < n.C; ++k)
    for (int c = 0; c < cg; ++c)
      for (int a = 0; a < n.kh; ++a)
        for (int b = 0; b < n.kw; ++b)
          w[(((size_t)k * n.kh + a) * n.kw + b) * cg + c] = s[(((size_t)k * cg + c) * n.kh + a) * n.kw + b];
  return w;
}

Loc tensor_loc(temco_plan_s* P, int id) { return P->loc.at(id); }

// ---------------------------------------------------------------------------
// lowering of one fused group into the SIMT interpreter's node table
// ---------------------------------------------------------------------------
struct GroupLowering {
  temco_plan_s* P;
  std::set<int> members;
  std::map<int, int> made;
  std::map<int, int> depth;   // expression depth of each lowered node (device recursion)

  int node(int v) {
    auto it = made.find(v);
    if (it != made.end()) return it->second;
    const IR& ir = P->ir;
    const Node& n = ir.nodes[v];
    GNode g{};
    g.C = n.C; g.H = n.H; g.W = n.W;
    g.w = g.b = -1;
    std::vector<int> kids;
    if (!members.count(v)) {
      g.op = G_EXT;
      g.t = tensor_loc(P, v);
      g.tC = n.C; g.tH = n.H; g.tW = n.W;
    } else if (n.role == ROLE_LCONV) {
      const int r = ir.oin[v][0];
      const Node& rn = ir.nodes[r];
      g.op = G_LCONV;
      g.R = rn.C;
      g.t = tensor_loc(P, r);
      g.tC = rn.C; g.tH = rn.H; g.tW = rn.W;
      g.w = push_params(P, n.w);
      g.b = push_params(P, n.b);
    } else {
      switch (n.op) {
        case OP_BN: {
          std::vector<float> sc, sh;
          bn_scale_shift(n, sc, sh);
          g.op = G_AFFINE;
          g.w = push_params(P, sc);
          g.b = push_params(P, sh);
          break;
        }
        case OP_RELU: g.op = G_RELU; break;
        case OP_SILU: g.op = G_SILU; break;
        case OP_ADD: g.op = G_ADD; break;
        case OP_CONCAT: g.op = G_CONCAT; break;
        case OP_MAXPOOL: g.op = G_MAXPOOL; g.k = n.kh; g.s = n.sh; g.p = n.ph; break;
        case OP_AVGPOOL: g.op = G_AVGPOOL; g.k = n.kh; g.s = n.sh; g.p = 0; break;
        default: throw std::runtime_error("unexpected op inside a fused group");
      }
      for (int i : ir.oin[v]) kids.push_back(node(i));
    }
    int d = 1;
    for (int k : kids) d = std::max(d, 1 + depth[k]);
    g.nin = (int)kids.size();
    g.child = (int)P->gchild_h.size();
    P->gchild_h.insert(P->gchild_h.end(), kids.begin(), kids.end());
    int id = (int)P->gnodes_h.size();
    P->gnodes_h.push_back(g);
    depth[id] = d;
    P->max_expr_depth = std::max(P->max_expr_depth, d);
    made[v] = id;
    return id;
  }
};

// ---------------------------------------------------------------------------
// arena: greedy best-offset placement of the schedule's tensors by lifetime
// ---------------------------------------------------------------------------
int64_t plan_arena(temco_plan_s* P) {
  const IR& ir = P->ir;
  const int T = (int)ir.steps.size();
  std::map<int, int> def, last;
  for (int t = 0; t < T; ++t) {
    std::vector<int> outs = {ir.steps[t].out};
    outs.insert(outs.end(), ir.steps[t].extra.begin(), ir.steps[t].extra.end());
    for (int o : outs) {
      def[o] = t;
      if (!last.count(o)) last[o] = t;
    }
    for (int x : ir.steps[t].in) last[x] = t;
  }
  struct Item { int id; int64_t bytes; int a, b; int64_t off; };
  std::vector<Item> items;
  const int64_t elem = P->bf16 ? 2 : 4;
  for (auto& kv : def) {
    int id = kv.first;
    if (id == ir.input || id == ir.output) continue;
    const Node& n = ir.nodes[id];
    int64_t bytes = (int64_t)ir.batch * n.C * n.H * n.W * elem;
    bytes = (bytes + 1023) / 1024 * 1024;
    items.push_back({id, bytes, kv.second, last[id], 0});
  }
  std::sort(items.begin(), items.end(), [](const Item& x, const Item& y) {
    return x.bytes != y.bytes ? x.bytes > y.bytes : x.id < y.id;
  });
  std::vector<Item> placed;
  int64_t total = 0;
  for (Item& it : items) {
    std::vector<std::pair<int64_t, int64_t>> busy;
    for (const Item& q : placed)
      if (!(q.b < it.a || it.b < q.a)) busy.push_back({q.off, q.off + q.bytes});
    std::sort(busy.begin(), busy.end());
    int64_t off = 0;
    for (auto& r : busy) {
      if (off + it.bytes <= r.first) break;
      off = std::max(off, r.second);
    }
    it.off = off;
    placed.push_back(it);
    total = std::max(total, off + it.bytes);
  }
  const int32_t dt = P->bf16 ? DT_BF16 : DT_F32;
  for (const Item& it : placed) P->loc[it.id] = Loc{W_ARENA, dt, it.off};
  P->loc[ir.input] = Loc{W_INPUT, dt, 0};
  P->loc[ir.output] = Loc{W_OUTPUT, DT_F32, 0};
  return total;
}

int64_t tensor_bytes(const temco_plan_s* P, int id) {
  const Node& n = P->ir.nodes[id];
  int64_t el = (int64_t)P->ir.batch * n.C * n.H * n.W;
  return el * (id == P->ir.output ? 4 : (P->bf16 ? 2 : 4));
}

// lowering of one fused-group step (one output) onto the fastest kernel that takes its shape
void lower_group(temco_plan_s* P, const Step& s, StepExec& e) {
  IR& ir = P->ir;
  const int N = ir.batch;
  const Node& v = ir.nodes[s.out];
  // groups with a 3x3/s2 max-pooled 64-channel member (the stem restore copies):
  // restore-once mma.sync kernel; single-input groups: the lean mma.sync kernels;
  // opt-in (TEMCO_FLAG_MMA_CAT, measured slower than tcgen05): the generic mma.sync
  // concat kernel; else tcgen05, else the interpreter
  const bool mma_ok = P->bf16 && !(P->flags & TEMCO_FLAG_SIMT_ONLY);
  std::vector<uint16_t> scratch;
  CatDesc cd;
  const bool cat_form = mma_ok && mma_cat_lower(ir, s, P->loc, scratch, cd);
  if (cat_form && mma_poolcat_ok(cd) && !getenv("TEMCO_NO_POOLCAT") &&
      mma_cat_lower(ir, s, P->loc, P->tcw_h, e.cat)) {
    e.kind = K_GROUP_CAT;
    e.kernel = "mma_poolcat";
    e.launches = 1;
    return;
  }
  if (mma_ok && ir.nodes[ir.oin[s.out][0]].C <= 256 &&
      mma_lower_chain(ir, s, P->loc, P->tcw_h, e.mma) &&
      ((P->flags & TEMCO_FLAG_MMA_SMALL) || (mma_lean_ok(e.mma) && !getenv("TEMCO_NO_LEAN")))) {
    e.kind = K_GROUP_MMA;
    e.kernel = mma_lean_ok(e.mma) ? "mma_lean" : "mma_chain";
    e.launches = 1;
    return;
  }
  if (cat_form && ((mma_catp_ok(cd) && !getenv("TEMCO_NO_CATP")) || (P->flags & TEMCO_FLAG_MMA_CAT)) &&
      mma_cat_lower(ir, s, P->loc, P->tcw_h, e.cat)) {
    e.kind = K_GROUP_CAT;
    e.kernel = mma_catp_ok(e.cat) ? "mma_catp" : "mma_cat";
    e.launches = 1;
    return;
  }
  // full-width residual chains with an fconv root: the CTA-pair tcgen05 kernel
  if (P->bf16 && !(P->flags & TEMCO_FLAG_SIMT_ONLY) &&
      pair::pair_lower_chain(ir, s, P->loc, P->tcw_h, P->params_h, e.pr)) {
    e.kind = K_GROUP_PAIR;
    e.kernel = "tc_pair";
    e.launches = 1;
    return;
  }
  if (P->bf16 && !(P->flags & TEMCO_FLAG_SIMT_ONLY) &&
      tc_lower_chain(ir, s, P->loc, P->tcw_h, P->params_h, e.tc)) {
    e.kind = K_GROUP_TC;
    e.kernel = "tc_chain";
    e.launches = 1;
    return;
  }
  // groups whose per-tile reduced inputs exceed shared memory: TMEM-resident levels
  if (P->bf16 && !(P->flags & TEMCO_FLAG_SIMT_ONLY) &&
      wide::tc_lower_chain(ir, s, P->loc, P->tcw_h, P->params_h, e.tcw)) {
    e.kind = K_GROUP_TCW;
    e.kernel = "tc_chain_wide";
    e.launches = 1;
    return;
  }
  GroupLowering gl{P, std::set<int>(s.members.begin(), s.members.end()), {}};
  GroupDesc& g = e.grp;
  int tsrc;
  if (v.role == ROLE_FCONV) {
    g.root = ROOT_FCONV;
    tsrc = ir.oin[s.out][0];
    g.Nout = v.C;
    if (v.C > 256) throw std::runtime_error("fused fconv with more than 256 outputs");
    g.F = push_params(P, v.w);
    g.Fb = push_params(P, v.b);
    gl.members.erase(s.out);
  } else if (v.op == OP_GAP) {
    g.root = ROOT_GAP;
    tsrc = ir.oin[s.out][0];
    gl.members.erase(s.out);
  } else {
    g.root = ROOT_STORE;
    tsrc = s.out;
  }
  const Node& tn = ir.nodes[tsrc];
  g.tnode = gl.node(tsrc);
  g.N = N; g.H = tn.H; g.W = tn.W; g.C = tn.C;
  g.y = tensor_loc(P, s.out);
  e.kind = K_GROUP_SIMT;
  e.kernel = g.root == ROOT_GAP ? "simt_group_gap" : "simt_group";
  e.launches = 1;
  return;
}

void lower(temco_plan_s* P) {
  IR& ir = P->ir;
  const int N = ir.batch;
  P->exec.assign(ir.steps.size(), StepExec());
  for (size_t t = 0; t < ir.steps.size(); ++t) {
    const Step& s = ir.steps[t];
    StepExec& e = P->exec[t];
    const Node& v = ir.nodes[s.out];
    for (int m : s.members) e.flops += node_flops(ir, m);
    for (int x : s.in) e.io_bytes += tensor_bytes(P, x);
    if (v.op != OP_INPUT) e.io_bytes += tensor_bytes(P, s.out);
    for (int x : s.extra) e.io_bytes += tensor_bytes(P, x);
    if (s.group && s.members.size() == 2 && ir.nodes[s.members[0]].op == OP_CONV &&
        ir.nodes[s.members[0]].groups > 1) {
      // CP depthwise core pair (reading R34): one kernel, the K x 1 output stays in registers
      const Node& v = ir.nodes[s.members[0]];
      const Node& h = ir.nodes[s.members[1]];
      const Node& x = ir.nodes[ir.oin[s.members[0]][0]];
      DwPairDesc& q = e.dwp;
      q = DwPairDesc{};
      q.x = tensor_loc(P, x.id);
      q.y = tensor_loc(P, s.out);
      q.N = N; q.H = x.H; q.W = x.W; q.C = x.C;
      q.H1 = v.H; q.Ho = h.H; q.Wo = h.W; q.K = v.kh;
      q.sv = v.sh; q.pv = v.ph; q.sh = h.sw; q.ph = h.pw;
      if (h.kw != v.kh || v.C != x.C) throw std::runtime_error("CP core pair: unexpected shapes");
      q.wv = push_params(P, v.w);
      q.wh = push_params(P, h.w);
      q.bv = push_params(P, v.b);
      q.bh = push_params(P, h.b);
      e.kind = K_DWPAIR;
      e.kernel = dwpair_fast_ok(q) ? "simt_dwpair" : "simt_dwpair_generic";
      e.launches = 1;
      continue;
    }
    if (s.group && !s.extra.empty()) {
      // merged group (reading R37): one CTA-pair launch computing every reduce output from one
      // restore when its kernel takes the shape; else the group replayed once per output
      std::vector<uint16_t> scratch;
      CatDesc cd;
      if (P->bf16 && !(P->flags & TEMCO_FLAG_SIMT_ONLY) && !getenv("TEMCO_NO_POOLCAT") &&
          mma_cat_lower(ir, s, P->loc, scratch, cd) && mma_poolcat_ok(cd) &&
          mma_cat_lower(ir, s, P->loc, P->tcw_h, e.cat)) {   // the restore-once pooled kernel, stacked F
        e.kind = K_GROUP_CAT;
        e.kernel = "mma_poolcat";
        e.launches = 1;
        continue;
      }
      if (P->bf16 && !(P->flags & TEMCO_FLAG_SIMT_ONLY) &&
          pair::pair_lower_chain(ir, s, P->loc, P->tcw_h, P->params_h, e.pr)) {
        e.kind = K_GROUP_PAIR;
        e.kernel = "tc_pair";
        e.launches = 1;
        continue;
      }
      e.kind = K_MULTI;
      e.launches = 0;
      std::vector<int> outs = {s.out};
      outs.insert(outs.end(), s.extra.begin(), s.extra.end());
      for (int o : outs) {
        Step sub;
        sub.out = o;
        sub.in = s.in;
        sub.group = true;
        for (int m : s.members)
          if (m == o || std::find(outs.begin(), outs.end(), m) == outs.end()) sub.members.push_back(m);
        StepExec se;
        lower_group(P, sub, se);
        if (e.kernel.empty() || e.kernel == se.kernel) e.kernel = se.kernel;
        else e.kernel = "multi";
        e.launches += se.launches;
        e.sub.push_back((int)P->sub_exec.size());
        P->sub_exec.push_back(std::move(se));
      }
      continue;
    }
    if (s.group) {
      lower_group(P, s, e);
      continue;
    }
    switch (v.op) {
      case OP_INPUT:
        e.kind = K_NONE;
        e.kernel = "none";
        break;
      case OP_CONV: {
        if (P->bf16 && !(P->flags & TEMCO_FLAG_SIMT_ONLY) && !getenv("TEMCO_NO_RKMMA") && v.groups == 1) {
          const Node& x = ir.nodes[ir.oin[s.out][0]];
          ConvDesc c{};
          c.x = tensor_loc(P, x.id);
          c.y = tensor_loc(P, s.out);
          c.N = N; c.H = x.H; c.W = x.W; c.C = x.C;
          c.Ho = v.H; c.Wo = v.W; c.K = v.C;
          c.kh = v.kh; c.kw = v.kw; c.sh = v.sh; c.sw = v.sw; c.ph = v.ph; c.pw = v.pw; c.groups = v.groups;
          c.b = v.b ? push_params(P, v.b) : -1;
          {   // reduced-rank cores: TMA-staged footprints, ldmatrix A / B, mma.sync (kernels_tile.cu)
            const std::vector<float> w = repack_conv(v, x.C);
            if (tile_conv_lower(c, w.data(), P->tcw_h, e.tile)) {
              e.kind = K_CONV_TILE;
              e.kernel = "mma_conv_tile";
              e.launches = 1;
              break;
            }
          }
          // 3x3 cores on 8 channels: the direct SIMT kernel measured faster (kernels_simt.cu)
          // (wider outputs stay on the tcgen05 implicit GEMM: measured faster for K > 64)
          if (c.C <= 256 && c.K <= 64 && !(c.C == 8 && c.K == 8 && c.kh * c.kw > 1)) {
            const std::vector<float> w = repack_conv(v, x.C);
            if (conv_rank_mma_lower(c, w.data(), P->tcw_h, e.rk)) {
              e.kind = K_CONV_RK;
              e.kernel = "mma_conv_rank";
              e.launches = 1;
              break;
            }
          }
        }
        const bool rank_conv = [&] {   // reduced-rank core conv: the memory-bound SIMT kernel
          if (!P->bf16 || getenv("TEMCO_CONV_TC")) return false;
          const Node& x = ir.nodes[ir.oin[s.out][0]];
          ConvDesc c{};
          c.x = tensor_loc(P, x.id);
          c.y = tensor_loc(P, s.out);
          c.N = N; c.H = x.H; c.W = x.W; c.C = x.C;
          c.Ho = v.H; c.Wo = v.W; c.K = v.C;
          c.kh = v.kh; c.kw = v.kw; c.sh = v.sh; c.sw = v.sw; c.ph = v.ph; c.pw = v.pw; c.groups = v.groups;
          return conv_rank_ok(c);
        }();
        if (!rank_conv && P->bf16 && !(P->flags & TEMCO_FLAG_SIMT_ONLY) && ir.nodes[ir.oin[s.out][0]].C % 8 == 0 &&
            conv_tc_lower(ir, s.out, P->loc, P->tcw_h, P->params_h, e.ctc)) {
          e.kind = K_CONV_TC;
          e.kernel = "tc_conv";
          e.launches = 1;
          break;
        }
        const Node& x = ir.nodes[ir.oin[s.out][0]];
        ConvDesc& c = e.conv;
        c.x = tensor_loc(P, x.id);
        c.y = tensor_loc(P, s.out);
        c.N = N; c.H = x.H; c.W = x.W; c.C = x.C;
        c.Ho = v.H; c.Wo = v.W; c.K = v.C;
        c.kh = v.kh; c.kw = v.kw; c.sh = v.sh; c.sw = v.sw; c.ph = v.ph; c.pw = v.pw; c.groups = v.groups;
        c.w = push_params(P, repack_conv(v, x.C));
        c.b = push_params(P, v.b);
        c.w2 = -1;
        if (v.groups == x.C && v.C == x.C) {   // depthwise: [tap][C] copy for the vectorised kernel
          std::vector<float> w2((size_t)v.kh * v.kw * v.C);
          const std::vector<float>& src = *v.w;
          for (int k = 0; k < v.C; ++k)
            for (int t = 0; t < v.kh * v.kw; ++t) w2[(size_t)t * v.C + k] = src[(size_t)k * v.kh * v.kw + t];
          c.w2 = push_params(P, w2);
        }
        e.kind = K_CONV;
        e.stem = !(P->flags & TEMCO_FLAG_SIMT_ONLY) && !dwconv_vec_ok(c) && !conv_rank_ok(c) && conv_stem_ok(c);
        e.kernel = e.stem ? "mma_conv_stem" : v.groups > 1 ? (dwconv_vec_ok(c) ? "simt_dwconv_vec" : "simt_dwconv") : conv_rank_ok(c) ? "simt_conv_rank" : conv_small_ok(c) ? "simt_conv_small" : "simt_conv";
        e.launches = 1;
        // a standalone 1x1 / stride-1 conv left to the generic SIMT kernel (the unfused restores and
        // reduces of the ablation plans, Cout > 256) is a plain NHWC GEMM y[NHW, O] = x[NHW, C] W^T:
        // cuBLAS, bf16 operands, fp32 accumulate; bf16 output written directly when there is no bias
        if (e.kernel == "simt_conv" && P->bf16 && !(P->flags & TEMCO_FLAG_SIMT_ONLY) && v.w &&
            v.kh == 1 && v.kw == 1 && v.sh == 1 && v.sw == 1 && v.ph == 0 && v.pw == 0 && v.groups == 1 &&
            c.x.dtype == DT_BF16 && c.y.dtype == DT_BF16 && x.C % 8 == 0 && v.C % 8 == 0 && !getenv("TEMCO_NO_CONV_BLAS")) {
          GemmDesc& g = e.gm;
          g = GemmDesc{};
          g.x = c.x;
          g.y = c.y;
          g.y2 = Loc{-1, 0, 0};
          g.M = N * x.H * x.W;
          g.K = x.C;
          g.O = v.C;
          g.relu = 0;
          if (gemm_lower(g, v.w->data(), v.b ? v.b.get() : nullptr, P->tcw_h, P->params_h, P->lin_ws_elems)) {
            e.kind = K_GEMM;
            e.kernel = "tc_gemm_conv1x1";
          }
        }
        break;
      }
      case OP_CONVT: {
        const Node& x = ir.nodes[ir.oin[s.out][0]];
        ConvDesc& c = e.conv;
        c.x = tensor_loc(P, x.id);
        c.y = tensor_loc(P, s.out);
        c.N = N; c.H = x.H; c.W = x.W; c.C = x.C;
        c.Ho = v.H; c.Wo = v.W; c.K = v.C;
        c.kh = v.kh; c.kw = v.kw; c.sh = v.sh; c.sw = v.sw; c.ph = v.ph; c.pw = v.pw; c.groups = 1;
        // W [C][K][kh][kw] (ConvTranspose2d layout) -> [kh*kw][K][C]
        std::vector<float> w((size_t)v.kh * v.kw * v.C * x.C);
        const std::vector<float>& src = *v.w;
        for (int ci = 0; ci < x.C; ++ci)
          for (int o = 0; o < v.C; ++o)
            for (int t = 0; t < v.kh * v.kw; ++t)
              w[((size_t)t * v.C + o) * x.C + ci] = src[((size_t)ci * v.C + o) * v.kh * v.kw + t];
        c.w = push_params(P, w);
        c.b = push_params(P, v.b);
        c.w2 = -1;
        e.kind = K_CONVT;
        e.kernel = "simt_conv_transpose";
        e.launches = 1;
        // k x k / stride k, no padding (the UNet up-conv): one GEMM x[NHW, C] W'[k*k*K, C]^T whose
        // epilogue stores column (i*k + j)*K + o at output pixel (h*k + i, w*k + j)
        if (P->bf16 && !(P->flags & TEMCO_FLAG_SIMT_ONLY) && v.kh == v.sh && v.kw == v.sw && v.kh == v.kw &&
            v.ph == 0 && v.pw == 0 && x.C % 8 == 0 && c.x.dtype == DT_BF16 && c.y.dtype == DT_BF16) {
          GemmDesc& g = e.gm;
          g = GemmDesc{};
          g.x = c.x;
          g.y = c.y;
          g.y2 = Loc{-1, 0, 0};
          g.M = N * x.H * x.W;
          g.K = x.C;
          g.O = v.kh * v.kw * v.C;
          g.shuffle_k = v.kh;
          g.sh_H = x.H; g.sh_W = x.W; g.sh_Co = v.C;
          std::vector<float> bias_t;
          if (v.b)
            for (int t = 0; t < v.kh * v.kw; ++t) bias_t.insert(bias_t.end(), v.b->begin(), v.b->end());
          if (gemm_lower(g, w.data(), v.b ? &bias_t : nullptr, P->tcw_h, P->params_h, P->lin_ws_elems)) {
            e.kind = K_GEMM;
            e.kernel = "tc_gemm_convt";
          }
        }
        break;
      }
      case OP_LINEAR: {
        const Node& x = ir.nodes[ir.oin[s.out][0]];
        LinearDesc& l = e.lin;
        l.x = tensor_loc(P, x.id);
        l.y = tensor_loc(P, s.out);
        l.N = N; l.K = x.C * x.H * x.W; l.O = v.C;
        // permute columns from NCHW flattening (c, h, w) to our NHWC (h, w, c)
        std::vector<float> w((size_t)l.O * l.K);
        const std::vector<float>& src = *v.w;
        for (int o = 0; o < l.O; ++o)
          for (int c = 0; c < x.C; ++c)
            for (int hw = 0; hw < x.H * x.W; ++hw)
              w[(size_t)o * l.K + (size_t)hw * x.C + c] = src[(size_t)o * l.K + (size_t)c * x.H * x.W + hw];
        l.w = push_params(P, w);
        l.b = push_params(P, v.b);
        l.relu = 0;
        e.kind = K_LINEAR;
        e.kernel = "simt_linear";
        if (P->bf16 && !(P->flags & TEMCO_FLAG_SIMT_ONLY) && l.x.dtype == DT_BF16) {
          // bf16 plans: the head is a GEMM on the tcgen05 kernel (fused bias; a following
          // standalone ReLU step is produced by the same epilogue as a second output)
          GemmDesc& g = e.gm;
          g = GemmDesc{};
          g.x = l.x;
          g.y = l.y;
          g.y2 = Loc{-1, 0, 0};
          g.M = l.N;
          g.K = l.K;
          g.O = l.O;
          g.relu = 0;
          if (gemm_lower(g, w.data(), v.b ? v.b.get() : nullptr, P->tcw_h, P->params_h, P->lin_ws_elems)) {
            e.kind = K_GEMM;
            e.kernel = "tc_gemm";
          }
        }
        e.launches = 1;
        break;
      }
      default: {
        EwDesc& d = e.ew;
        const Node& x = ir.nodes[ir.oin[s.out][0]];
        d.y = tensor_loc(P, s.out);
        d.N = N; d.H = x.H; d.W = x.W; d.C = v.C; d.Ho = v.H; d.Wo = v.W;
        d.n_in = (int)ir.oin[s.out].size();
        if (d.n_in > kMaxEwInputs) throw std::runtime_error("too many inputs for a standalone op");
        for (int j = 0; j < d.n_in; ++j) {
          d.x[j] = tensor_loc(P, ir.oin[s.out][j]);
          d.xc[j] = ir.nodes[ir.oin[s.out][j]].C;
        }
        d.scale = d.shift = -1;
        switch (v.op) {
          case OP_BN: {
            std::vector<float> sc, sh;
            bn_scale_shift(v, sc, sh);
            d.kind = EW_BN;
            d.scale = push_params(P, sc);
            d.shift = push_params(P, sh);
            break;
          }
          case OP_RELU: d.kind = EW_RELU; break;
          case OP_SILU: d.kind = EW_SILU; break;
          case OP_ADD: d.kind = EW_ADD; break;
          case OP_CONCAT: d.kind = EW_CONCAT; break;
          case OP_MAXPOOL: d.kind = EW_MAXPOOL; d.k = v.kh; d.s = v.sh; d.p = v.ph; break;
          case OP_AVGPOOL: d.kind = EW_AVGPOOL; d.k = v.kh; d.s = v.sh; d.p = 0; break;
          case OP_GAP: d.kind = EW_GAP; break;
          default: throw std::runtime_error("unexpected standalone op");
        }
        e.kind = K_EW;
        e.kernel = std::string("simt_") + op_name(v.op);
        e.launches = 1;
      }
    }
  }
  // a standalone ReLU right after a GEMM head layer (AlexNet / VGG FC stacks): the GEMM
  // epilogue writes it as a second output, the ReLU step launches nothing
  for (size_t t = 0; t + 1 < ir.steps.size(); ++t) {
    StepExec& e = P->exec[t];
    StepExec& r = P->exec[t + 1];
    const Step& s1 = ir.steps[t + 1];
    if (e.kind != K_GEMM || e.gm.shuffle_k || e.gm.relu || r.kind != K_EW || s1.group) continue;
    if (ir.nodes[s1.out].op != OP_RELU || ir.oin[s1.out].size() != 1 || ir.oin[s1.out][0] != ir.steps[t].out) continue;
    e.gm.y2 = tensor_loc(P, s1.out);
    r.kind = K_NONE;
    r.kernel = "in_gemm";
    r.launches = 0;
  }
}

void json_ints(std::ostringstream& o, const std::vector<int>& v) {
  o << "[";
  for (size_t i = 0; i < v.size(); ++i) o << (i ? "," : "") << v[i];
  o << "]";
}

std::string make_json(const temco_plan_s* P) {
  const IR& ir = P->ir;
  std::ostringstream o;
  int launches = 0;
  for (auto& e : P->exec) launches += e.launches;
  o << "{\"peak_fused\":" << ir.peak_fused << ",\"peak_unfused\":" << ir.peak_unfused
    << ",\"arena_bytes\":" << P->arena_bytes << ",\"n_L\":" << ir.nL << ",\"n_O\":" << ir.O.size()
    << ",\"launches\":" << launches << ",\"dtype\":\"" << (P->bf16 ? "bf16" : "f32") << "\",\"decisions\":[";
  for (size_t i = 0; i < ir.decisions.size(); ++i) {
    const SkipDecision& d = ir.decisions[i];
    o << (i ? "," : "") << "{\"node\":" << d.node << ",\"kind\":\""
      << (d.kind == 0 ? "skip-optimized" : d.kind == 1 ? "skip-unreducible" : "skip-rejected") << "\",\"list\":";
    json_ints(o, d.list);
    o << "}";
  }
  o << "],\"O\":";
  json_ints(o, ir.O);
  o << ",\"steps\":[";
  for (size_t t = 0; t < ir.steps.size(); ++t) {
    const Step& s = ir.steps[t];
    const Node& v = ir.nodes[s.out];
    o << (t ? "," : "") << "{\"kind\":\"" << (s.group ? "group" : "op") << "\",\"out\":" << s.out << ",\"op\":\""
      << op_name(v.op) << "\",\"role\":\"" << role_name(v.role) << "\",\"members\":";
    json_ints(o, s.members);
    o << ",\"inputs\":";
    json_ints(o, s.in);
    o << ",\"bytes\":" << ir.size(s.out) << ",\"extra\":";
    json_ints(o, s.extra);
    // shapes [C, H, W] of the step's inputs and output (per image)
    o << ",\"in_chw\":[";
    for (size_t i = 0; i < s.in.size(); ++i) {
      const Node& x = ir.nodes[s.in[i]];
      o << (i ? "," : "") << "[" << x.C << "," << x.H << "," << x.W << "]";
    }
    o << "],\"out_chw\":[" << v.C << "," << v.H << "," << v.W << "]";
    if (!P->exec.empty()) {
      const StepExec& e = P->exec[t];
      o << ",\"kernel\":\"" << e.kernel << "\",\"flops\":" << e.flops << ",\"io_bytes\":" << e.io_bytes
        << ",\"launches\":" << e.launches;
      if (e.kind == K_GROUP_TC)
        o << ",\"alg_flops\":" << e.tc.alg_flops << ",\"alg_bytes\":" << e.tc.alg_bytes << ",\"tc\":{\"n_prod\":"
          << e.tc.n_prod << ",\"n_mma\":" << e.tc.n_mma << ",\"units\":" << e.tc.units << ",\"stages\":" << e.tc.stages
          << ",\"resident\":" << e.tc.resident << ",\"smem\":" << e.tc.smem_bytes << ",\"tmem\":" << e.tc.tmem_cols << ",\"fres\":" << e.tc.fres << ",\"slots\":" << e.tc.ns << ",\"ntiles\":"
          << e.tc.ntiles << ",\"Cc\":" << e.tc.Cc << ",\"levels\":" << e.tc.n_levels << "}";
      if (e.kind == K_GROUP_TCW)
        o << ",\"alg_flops\":" << e.tcw.alg_flops << ",\"alg_bytes\":" << e.tcw.alg_bytes << ",\"tc\":{\"variant\":\"wide\",\"n_prod\":"
          << e.tcw.n_prod << ",\"n_mma\":" << e.tcw.n_mma << ",\"units\":" << e.tcw.units << ",\"stages\":" << e.tcw.stages
          << ",\"resident\":" << e.tcw.resident << ",\"smem\":" << e.tcw.smem_bytes << ",\"tmem\":" << e.tcw.tmem_cols
          << ",\"ntiles\":" << e.tcw.ntiles << ",\"Cc\":" << e.tcw.Cc << ",\"levels\":" << e.tcw.n_levels << "}";
      if (e.kind == K_GROUP_PAIR)
        o << ",\"alg_flops\":" << e.pr.alg_flops << ",\"alg_bytes\":" << e.pr.alg_bytes << ",\"tc\":{\"variant\":\"pair\",\"stages\":"
          << e.pr.stages << ",\"slot\":" << e.pr.slot << ",\"resident\":" << e.pr.resident << ",\"smem\":" << e.pr.smem_bytes << ",\"ntiles\":" << e.pr.ntiles << ",\"units\":" << e.pr.nunits
          << ",\"levels\":" << e.pr.n_levels << ",\"terms\":" << e.pr.n_terms << "}";
      if (e.kind == K_GEMM) o << ",\"alg_flops\":" << e.gm.alg_flops << ",\"alg_bytes\":" << e.gm.alg_bytes << ",\"splits\":" << e.gm.splits;
      if (e.kind == K_CONV_TC) o << ",\"alg_flops\":" << e.ctc.alg_flops << ",\"alg_bytes\":" << e.ctc.alg_bytes;
      if (e.kind == K_CONV_RK) o << ",\"alg_flops\":" << e.rk.alg_flops << ",\"alg_bytes\":" << e.rk.alg_bytes;
      if (e.kind == K_CONV_TILE) o << ",\"alg_flops\":" << e.tile.alg_flops << ",\"alg_bytes\":" << e.tile.alg_bytes;
      if (e.kind == K_GROUP_CAT) o << ",\"alg_flops\":" << e.cat.alg_flops << ",\"alg_bytes\":" << e.cat.alg_bytes;
      if (e.kind == K_GROUP_MMA) o << ",\"alg_flops\":" << e.mma.alg_flops << ",\"alg_bytes\":" << e.mma.alg_bytes;
    }
    o << ",\"live\":" << ir.live_fused[t] << "}";
  }
  o << "],\"live_unfused\":[";
  for (size_t t = 0; t < ir.live_unfused.size(); ++t) o << (t ? "," : "") << ir.live_unfused[t];
  o << "]}";
  return o.str();
}

template <class T>
temco_status upload(T** dst, const std::vector<T>& src) {
  if (src.empty()) return TEMCO_OK;
  if (cudaMalloc(dst, src.size() * sizeof(T)) != cudaSuccess) return set_err(TEMCO_ERR_OUT_OF_MEMORY, "cudaMalloc");
  CUDA_TRY(cudaMemcpy(*dst, src.data(), src.size() * sizeof(T), cudaMemcpyHostToDevice));
  return TEMCO_OK;
}

void free_device(temco_plan_s* P) {
  for (auto& g : P->graphs)
    if (g.exec) cudaGraphExecDestroy(g.exec);
  cudaFree(P->params_d);
  cudaFree(P->gnodes_d);
  cudaFree(P->gchild_d);
  cudaFree(P->tcw_d);
  cudaFree(P->arena_d);
  cudaFree(P->host_in_d);
  cudaFree(P->host_out_d);
  for (int b = 0; b < 2; ++b) {
    cudaFree(P->async_in_d[b]);
    cudaFree(P->async_out_d[b]);
    if (P->ev_in_ready[b]) cudaEventDestroy(P->ev_in_ready[b]);
    if (P->ev_buf_free[b]) cudaEventDestroy(P->ev_buf_free[b]);
  }
  if (P->copy_stream) cudaStreamDestroy(P->copy_stream);
  cudaFree(P->lin_ws_d);
}

}  // namespace

bool temco::pdl_enabled() {
  static const bool on = getenv("TEMCO_NO_PDL") == nullptr;
  return on;
}

namespace {

RunPtrs run_ptrs(temco_plan_s* P, const void* in, void* out) {
  return RunPtrs{P->arena_d, in, out, P->params_d};
}

void launch_exec(temco_plan_s* P, const StepExec& e, const RunPtrs& rp, cudaStream_t st) {
  switch (e.kind) {
    case K_NONE: break;
    case K_CONVT: launch_conv_transpose(e.conv, rp, st); break;
    case K_DWPAIR: launch_dwpair(e.dwp, rp, st); break;
    case K_CONV:
      if (e.stem)
        launch_conv_stem(e.conv, rp, st);
      else if (dwconv_vec_ok(e.conv))
        launch_dwconv_vec(e.conv, rp, st);
      else if (conv_rank_ok(e.conv))
        launch_conv_rank(e.conv, rp, st);
      else if (conv_small_ok(e.conv))
        launch_conv_small(e.conv, rp, st);
      else
        launch_conv(e.conv, rp, st);
      break;
    case K_EW: launch_ew(e.ew, rp, st); break;
    case K_LINEAR: launch_linear(e.lin, rp, st); break;
    case K_GROUP_SIMT: launch_group_simt(e.grp, P->gnodes_d, P->gchild_d, rp, st); break;
    case K_GROUP_TC: launch_tc_chain(e.tc, P->tcw_d, rp, st); break;
    case K_GROUP_TCW: wide::launch_tc_chain(e.tcw, P->tcw_d, rp, st); break;
    case K_GROUP_PAIR: pair::launch_pair_chain(e.pr, rp, st); break;
    case K_GEMM: launch_gemm(e.gm, rp, P->lin_ws_d, st); break;
    case K_CONV_TC: launch_conv_tc(e.ctc, rp, st); break;
    case K_CONV_RK: launch_conv_rank_mma(e.rk, P->tcw_d, rp, st); break;
    case K_CONV_TILE: launch_tile_conv(e.tile, P->tcw_d, rp, st); break;
    case K_GROUP_CAT: launch_mma_cat(e.cat, P->tcw_d, rp, st); break;
    case K_GROUP_MMA: launch_mma_chain(e.mma, P->tcw_d, rp, st); break;
    case K_MULTI:
      for (int k : e.sub) launch_exec(P, P->sub_exec[k], rp, st);
      break;
  }
}

temco_status enqueue(temco_plan_s* P, const void* in, void* out, cudaStream_t st, cudaEvent_t* ev,
                     int64_t last_step = -1) {
  RunPtrs rp = run_ptrs(P, in, out);
  const size_t nsteps = last_step >= 0 ? (size_t)last_step + 1 : P->exec.size();
  for (size_t t = 0; t < nsteps; ++t) {
    const StepExec& e = P->exec[t];
    if (ev) CUDA_TRY(cudaEventRecord(ev[2 * t], st));
    launch_exec(P, e, rp, st);
    if (ev) CUDA_TRY(cudaEventRecord(ev[2 * t + 1], st));
  }
  cudaError_t err = cudaGetLastError();
  if (err != cudaSuccess) return set_err(TEMCO_ERR_CUDA, std::string("kernel launch: ") + cudaGetErrorString(err));
  return TEMCO_OK;
}

temco_status check_device(temco_plan_s* P) {
  if (!P) return set_err(TEMCO_ERR_INVALID_ARGUMENT, "plan is NULL");
  if (!P->has_device) return set_err(TEMCO_ERR_NO_DEVICE, "plan was created without a device");
  int dev = -1;
  CUDA_TRY(cudaGetDevice(&dev));
  if (dev != P->device) return set_err(TEMCO_ERR_DEVICE_MISMATCH, "current device differs from the plan's");
  return TEMCO_OK;
}

}  // namespace

extern "C" {

const char* temco_status_string(temco_status s) {
  switch (s) {
    case TEMCO_OK: return "ok";
    case TEMCO_ERR_INVALID_ARGUMENT: return "invalid argument";
    case TEMCO_ERR_INVALID_GRAPH: return "invalid graph";
    case TEMCO_ERR_UNSUPPORTED: return "unsupported";
    case TEMCO_ERR_OUT_OF_MEMORY: return "out of memory";
    case TEMCO_ERR_CUDA: return "cuda error";
    case TEMCO_ERR_DEVICE_MISMATCH: return "device mismatch";
    case TEMCO_ERR_NO_DEVICE: return "no device";
  }
  return "unknown status";
}

const char* temco_last_error(void) { return g_last_error.c_str(); }

temco_status temco_plan_create(const temco_layer* layers, int32_t n_layers, const temco_decomp* decomps,
                               int32_t n_decomps, const temco_edge* skip_edges, int32_t n_skip_edges,
                               const temco_config* cfg, temco_plan_t* out_plan) {
  if (!cfg || !out_plan) return set_err(TEMCO_ERR_INVALID_ARGUMENT, "cfg / out_plan is NULL");
  *out_plan = nullptr;
  if (cfg->dtype != TEMCO_F32 && cfg->dtype != TEMCO_BF16) return set_err(TEMCO_ERR_INVALID_ARGUMENT, "bad dtype");
  if ((cfg->flags & TEMCO_FLAG_OVERHEAD_ALWAYS) && (cfg->flags & TEMCO_FLAG_OVERHEAD_NEVER))
    return set_err(TEMCO_ERR_INVALID_ARGUMENT, "contradictory overhead flags");
  auto* P = new (std::nothrow) temco_plan_s();
  if (!P) return set_err(TEMCO_ERR_OUT_OF_MEMORY, "host allocation");
  P->cfg = *cfg;
  P->bf16 = cfg->dtype == TEMCO_BF16;
  P->flags = cfg->flags;
  BuildOptions opt;
  opt.distance_threshold = cfg->distance_threshold > 0 ? cfg->distance_threshold : 1;
  opt.skip_opt = !(cfg->flags & TEMCO_FLAG_NO_SKIPOPT);
  opt.fusion = !(cfg->flags & TEMCO_FLAG_NO_FUSION);
  opt.extensions = !(cfg->flags & TEMCO_FLAG_PAPER_SCHEDULE);
  opt.cse = !(cfg->flags & TEMCO_FLAG_NO_CSE);
  opt.cse_policy = (cfg->flags & TEMCO_FLAG_CSE_BOUND) ? 1 : 0;
  opt.reorder = !(cfg->flags & TEMCO_FLAG_NO_RESCHEDULE);
  opt.overhead_policy = (cfg->flags & TEMCO_FLAG_OVERHEAD_ALWAYS) ? 1 : (cfg->flags & TEMCO_FLAG_OVERHEAD_NEVER) ? 2 : 0;
  opt.bf16 = P->bf16;
  std::string err;
  temco_status st = build_ir(layers, n_layers, decomps, n_decomps, skip_edges, n_skip_edges, *cfg, opt, P->ir, err);
  if (st != TEMCO_OK) {
    delete P;
    return set_err(st, err);
  }
  const Node& on = P->ir.nodes[P->ir.output];
  if (on.H == 1 && on.W == 1 && (on.op == OP_LINEAR || on.op == OP_GAP)) {
    P->out_ndim = 2;
    P->out_dims[0] = cfg->batch;
    P->out_dims[1] = on.C;
  } else {
    P->out_ndim = 4;
    P->out_dims[0] = cfg->batch; P->out_dims[1] = on.H; P->out_dims[2] = on.W; P->out_dims[3] = on.C;
  }
  P->in_bytes = (int64_t)cfg->batch * cfg->height * cfg->width * cfg->channels * (P->bf16 ? 2 : 4);
  P->out_bytes = (int64_t)cfg->batch * on.C * on.H * on.W * 4;
  try {
    P->arena_bytes = plan_arena(P);
    lower(P);
  } catch (const std::exception& ex) {
    delete P;
    return set_err(TEMCO_ERR_UNSUPPORTED, std::string("lowering: ") + ex.what());
  }
  P->json = make_json(P);
  if (!(cfg->flags & TEMCO_FLAG_NO_DEVICE)) {
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess) {
      delete P;
      return set_err(TEMCO_ERR_NO_DEVICE, "no CUDA device (use TEMCO_FLAG_NO_DEVICE for host-only plans)");
    }
    P->device = dev;
    P->has_device = true;
    // the SIMT group interpreter recurses once per expression level (~128 B
    // frames, see -Xptxas -v); grow the per-thread stack when needed
    size_t need = 1024 + (size_t)P->max_expr_depth * 192, cur = 0;
    if (cudaDeviceGetLimit(&cur, cudaLimitStackSize) == cudaSuccess && cur < need &&
        cudaDeviceSetLimit(cudaLimitStackSize, need) != cudaSuccess) {
      delete P;
      return set_err(TEMCO_ERR_CUDA, "cudaDeviceSetLimit(cudaLimitStackSize)");
    }
    temco_status s2 = TEMCO_OK;
    if ((s2 = upload(&P->params_d, P->params_h)) != TEMCO_OK || (s2 = upload(&P->gnodes_d, P->gnodes_h)) != TEMCO_OK ||
        (s2 = upload(&P->gchild_d, P->gchild_h)) != TEMCO_OK || (s2 = upload(&P->tcw_d, P->tcw_h)) != TEMCO_OK) {
      free_device(P);
      delete P;
      return s2;
    }
    if (P->arena_bytes > 0 && cudaMalloc(&P->arena_d, P->arena_bytes) != cudaSuccess) {
      free_device(P);
      delete P;
      return set_err(TEMCO_ERR_OUT_OF_MEMORY, "arena cudaMalloc");
    }
    if (P->lin_ws_elems > 0) {
      if (cudaMalloc(&P->lin_ws_d, P->lin_ws_elems * sizeof(float)) != cudaSuccess) {
        free_device(P);
        delete P;
        return set_err(TEMCO_ERR_OUT_OF_MEMORY, "GEMM workspace cudaMalloc");
      }
    }
    std::string terr;
    std::vector<StepExec*> ex;   // every launch: the steps' and the replayed merged groups'
    for (auto& e : P->exec) ex.push_back(&e);
    for (auto& e : P->sub_exec) ex.push_back(&e);
    for (StepExec* e : ex)
      if (e->kind == K_CONV_TC && (!conv_tc_finalize(e->ctc, P->tcw_d, terr) ||
                                    !conv_tc_finalize_x(e->ctc, P->arena_d + e->ctc.x.off, terr))) {
        free_device(P);
        delete P;
        return set_err(TEMCO_ERR_CUDA, "tensor maps: " + terr);
      }
    if (!tc_finalize(ex.size(), [&](size_t i) -> TcChainDesc* {
          return ex[i]->kind == K_GROUP_TC ? &ex[i]->tc : nullptr;
        }, P->arena_d, P->tcw_d, terr)) {
      free_device(P);
      delete P;
      return set_err(TEMCO_ERR_CUDA, "tensor maps: " + terr);
    }
    if (!wide::tc_finalize(ex.size(), [&](size_t i) -> wide::TcChainDesc* {
          return ex[i]->kind == K_GROUP_TCW ? &ex[i]->tcw : nullptr;
        }, P->arena_d, P->tcw_d, terr)) {
      free_device(P);
      delete P;
      return set_err(TEMCO_ERR_CUDA, "tensor maps: " + terr);
    }
    for (StepExec* e : ex)
      if (e->kind == K_CONV_TILE && !tile_conv_finalize(e->tile, P->arena_d, terr)) {
        free_device(P);
        delete P;
        return set_err(TEMCO_ERR_CUDA, "tensor maps: " + terr);
      }
    for (StepExec* e : ex)
      if (e->kind == K_GEMM && !gemm_finalize(e->gm, P->arena_d, P->tcw_d, terr)) {
        free_device(P);
        delete P;
        return set_err(TEMCO_ERR_CUDA, "tensor maps: " + terr);
      }
    if (!pair::pair_finalize(ex.size(), [&](size_t i) -> pair::PairDesc* {
          return ex[i]->kind == K_GROUP_PAIR ? &ex[i]->pr : nullptr;
        }, P->arena_d, P->tcw_d, terr)) {
      free_device(P);
      delete P;
      return set_err(TEMCO_ERR_CUDA, "tensor maps: " + terr);
    }
  }
  // the host copies of large pools are no longer needed
  *out_plan = P;
  return TEMCO_OK;
}

temco_status temco_run(temco_plan_t P, const void* input, void* output, temco_stream_t stream) {
  temco_status st = check_device(P);
  if (st != TEMCO_OK) return st;
  if (!input || !output) return set_err(TEMCO_ERR_INVALID_ARGUMENT, "input / output is NULL");
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  if ((P->flags & TEMCO_FLAG_CUDA_GRAPH) && s != nullptr) {
    temco_plan_s::GraphEntry* g = nullptr;
    for (auto& e : P->graphs)
      if (e.exec && e.in == input && e.out == output && e.stream == s) g = &e;
    if (!g) {   // capture into the least recently used entry
      g = P->graphs[0].used <= P->graphs[1].used ? &P->graphs[0] : &P->graphs[1];
      if (g->exec) cudaGraphExecDestroy(g->exec);
      g->exec = nullptr;
      cudaGraph_t graph;
      CUDA_TRY(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
      temco_status e = enqueue(P, input, output, s, nullptr);
      cudaError_t ce = cudaStreamEndCapture(s, &graph);
      if (e != TEMCO_OK) return e;
      if (ce != cudaSuccess) return set_err(TEMCO_ERR_CUDA, std::string("capture: ") + cudaGetErrorString(ce));
      ce = cudaGraphInstantiate(&g->exec, graph, 0);
      cudaGraphDestroy(graph);
      if (ce != cudaSuccess) return set_err(TEMCO_ERR_CUDA, std::string("instantiate: ") + cudaGetErrorString(ce));
      g->in = input;
      g->out = output;
      g->stream = s;
    }
    g->used = ++P->graph_clock;
    CUDA_TRY(cudaGraphLaunch(g->exec, s));
    return TEMCO_OK;
  }
  return enqueue(P, input, output, s, nullptr);
}

temco_status temco_run_host(temco_plan_t P, const void* host_input, void* host_output, temco_stream_t stream) {
  temco_status st = check_device(P);
  if (st != TEMCO_OK) return st;
  if (!host_input || !host_output) return set_err(TEMCO_ERR_INVALID_ARGUMENT, "host buffers are NULL");
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  if (!P->host_in_d || !P->host_out_d) {
    cudaFree(P->host_in_d);
    cudaFree(P->host_out_d);
    P->host_in_d = P->host_out_d = nullptr;
    if (cudaMalloc(&P->host_in_d, P->in_bytes) != cudaSuccess || cudaMalloc(&P->host_out_d, P->out_bytes) != cudaSuccess) {
      cudaFree(P->host_in_d);   // all or nothing: a later call retries from scratch
      P->host_in_d = nullptr;
      P->host_out_d = nullptr;
      return set_err(TEMCO_ERR_OUT_OF_MEMORY, "staging buffers");
    }
  }
  CUDA_TRY(cudaMemcpyAsync(P->host_in_d, host_input, P->in_bytes, cudaMemcpyHostToDevice, s));
  st = temco_run(P, P->host_in_d, P->host_out_d, stream);
  if (st != TEMCO_OK) return st;
  CUDA_TRY(cudaMemcpyAsync(host_output, P->host_out_d, P->out_bytes, cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaStreamSynchronize(s));
  return TEMCO_OK;
}

temco_status temco_run_host_async(temco_plan_t P, const void* host_input, void* host_output,
                                  temco_stream_t stream) {
  temco_status st = check_device(P);
  if (st != TEMCO_OK) return st;
  if (!host_input || !host_output) return set_err(TEMCO_ERR_INVALID_ARGUMENT, "host buffers are NULL");
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  if (!P->copy_stream) {
    // all or nothing: on any failure release what was made, so a later call starts over
    auto release = [P]() {
      for (int b = 0; b < 2; ++b) {
        cudaFree(P->async_in_d[b]);
        cudaFree(P->async_out_d[b]);
        P->async_in_d[b] = P->async_out_d[b] = nullptr;
        if (P->ev_in_ready[b]) cudaEventDestroy(P->ev_in_ready[b]);
        if (P->ev_buf_free[b]) cudaEventDestroy(P->ev_buf_free[b]);
        P->ev_in_ready[b] = P->ev_buf_free[b] = nullptr;
      }
    };
    bool ok = true;
    for (int b = 0; b < 2 && ok; ++b)
      ok = cudaMalloc(&P->async_in_d[b], P->in_bytes) == cudaSuccess &&
           cudaMalloc(&P->async_out_d[b], P->out_bytes) == cudaSuccess;
    for (int b = 0; b < 2 && ok; ++b)
      ok = cudaEventCreateWithFlags(&P->ev_in_ready[b], cudaEventDisableTiming) == cudaSuccess &&
           cudaEventCreateWithFlags(&P->ev_buf_free[b], cudaEventDisableTiming) == cudaSuccess;
    cudaStream_t cs = nullptr;
    if (ok) ok = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking) == cudaSuccess;
    if (!ok) {
      release();
      return set_err(TEMCO_ERR_OUT_OF_MEMORY, "async staging buffers / events / copy stream");
    }
    P->copy_stream = cs;
  }
  const int b = P->async_flip;
  P->async_flip ^= 1;
  // staging buffer b is free once the run that read it (two calls ago) is done
  CUDA_TRY(cudaStreamWaitEvent(P->copy_stream, P->ev_buf_free[b], 0));
  CUDA_TRY(cudaMemcpyAsync(P->async_in_d[b], host_input, P->in_bytes, cudaMemcpyHostToDevice, P->copy_stream));
  CUDA_TRY(cudaEventRecord(P->ev_in_ready[b], P->copy_stream));
  CUDA_TRY(cudaStreamWaitEvent(s, P->ev_in_ready[b], 0));
  st = temco_run(P, P->async_in_d[b], P->async_out_d[b], stream);
  if (st != TEMCO_OK) return st;
  CUDA_TRY(cudaEventRecord(P->ev_buf_free[b], s));
  CUDA_TRY(cudaMemcpyAsync(host_output, P->async_out_d[b], P->out_bytes, cudaMemcpyDeviceToHost, s));
  return TEMCO_OK;
}

temco_status temco_run_profiled(temco_plan_t P, const void* input, void* output, temco_stream_t stream,
                                float* step_ms, int32_t n_steps) {
  temco_status st = check_device(P);
  if (st != TEMCO_OK) return st;
  if (!input || !output || !step_ms || n_steps != (int32_t)P->exec.size())
    return set_err(TEMCO_ERR_INVALID_ARGUMENT, "bad profiling arguments");
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  std::vector<cudaEvent_t> ev(2 * P->exec.size());
  for (auto& e : ev) CUDA_TRY(cudaEventCreate(&e));
  st = enqueue(P, input, output, s, ev.data());
  if (st == TEMCO_OK) {
    CUDA_TRY(cudaStreamSynchronize(s));
    for (size_t t = 0; t < P->exec.size(); ++t) cudaEventElapsedTime(&step_ms[t], ev[2 * t], ev[2 * t + 1]);
  }
  for (auto& e : ev) cudaEventDestroy(e);
  return st;
}

temco_status temco_debug_step_tensor(temco_plan_t P, const void* input, void* output, temco_stream_t stream,
                                     int32_t step, int32_t which, void* host_dst, int64_t capacity, int64_t* bytes) {
  temco_status st = check_device(P);
  if (st != TEMCO_OK) return st;
  if (!input || !output || !bytes || step < 0 || step >= (int32_t)P->exec.size() || which < 0 ||
      which > (int32_t)P->ir.steps[step].extra.size())
    return set_err(TEMCO_ERR_INVALID_ARGUMENT, "bad step-output arguments");
  const int id = which == 0 ? P->ir.steps[step].out : P->ir.steps[step].extra[which - 1];
  const Loc l = P->loc.count(id) ? P->loc.at(id) : Loc{W_INPUT, 0, 0};
  const int64_t need = tensor_bytes(P, id);
  *bytes = need;
  if (!host_dst) return TEMCO_OK;   // size query
  if (capacity < need) return set_err(TEMCO_ERR_INVALID_ARGUMENT, "host buffer too small for the step output");
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  st = enqueue(P, input, output, s, nullptr, step);
  if (st != TEMCO_OK) return st;
  const void* src = loc_ptr(l, run_ptrs(P, input, output));
  CUDA_TRY(cudaMemcpyAsync(host_dst, src, need, cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaStreamSynchronize(s));
  return TEMCO_OK;
}

temco_status temco_debug_step_output(temco_plan_t P, const void* input, void* output, temco_stream_t stream,
                                     int32_t step, void* host_dst, int64_t capacity, int64_t* bytes) {
  return temco_debug_step_tensor(P, input, output, stream, step, 0, host_dst, capacity, bytes);
}

temco_status temco_peak_internal_bytes(temco_plan_t P, int32_t which, int64_t* bytes) {
  if (!P || !bytes || (which != 0 && which != 1)) return set_err(TEMCO_ERR_INVALID_ARGUMENT, "bad arguments");
  *bytes = which == 0 ? P->ir.peak_fused : P->ir.peak_unfused;
  return TEMCO_OK;
}

temco_status temco_output_shape(temco_plan_t P, int64_t dims[4], int32_t* ndim) {
  if (!P || !dims || !ndim) return set_err(TEMCO_ERR_INVALID_ARGUMENT, "bad arguments");
  for (int i = 0; i < 4; ++i) dims[i] = P->out_dims[i];
  *ndim = P->out_ndim;
  return TEMCO_OK;
}

temco_status temco_plan_describe(temco_plan_t P, char* buf, size_t cap, size_t* needed) {
  if (!P) return set_err(TEMCO_ERR_INVALID_ARGUMENT, "plan is NULL");
  if (needed) *needed = P->json.size() + 1;
  if (buf && cap > 0) {
    size_t n = std::min(cap - 1, P->json.size());
    memcpy(buf, P->json.data(), n);
    buf[n] = 0;
  }
  return TEMCO_OK;
}

temco_status temco_plan_destroy(temco_plan_t P) {
  if (!P) return TEMCO_OK;
  if (P->has_device) free_device(P);
  delete P;
  return TEMCO_OK;
}

}  // extern "C"
