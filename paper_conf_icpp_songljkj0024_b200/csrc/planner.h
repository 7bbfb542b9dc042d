// Host-side TeMCO planner: decomposition expansion, liveness, skip connection
// optimization (Alg. 1/2), DCE, fusion grouping and peak accounting.
// Independent of the oracle (oracle/); both follow PAPER.md and the readings
// listed in DESIGN.md, and tests/test_plan_parity.py diffs the two.
#pragma once

#include <cstdint>
#include <map>
#include <memory>
#include <string>
#include <vector>

#include "../../include/temco.h"

namespace temco {

enum Op { OP_INPUT, OP_CONV, OP_BN, OP_RELU, OP_SILU, OP_ADD, OP_CONCAT, OP_MAXPOOL, OP_AVGPOOL, OP_GAP, OP_LINEAR,
          OP_CONVT /* transposed conv (UNet up-conv core) */ };
enum Role { ROLE_NONE, ROLE_FCONV, ROLE_CORE, ROLE_LCONV };

const char* op_name(Op op);
const char* role_name(Role r);

using Buf = std::shared_ptr<const std::vector<float>>;

struct Node {
  int id = -1;
  Op op = OP_INPUT;
  Role role = ROLE_NONE;
  int orig = -1;                 // original layer index
  std::vector<int> in;           // inputs in L (copies: inputs at creation)
  int kh = 1, kw = 1, sh = 1, sw = 1, ph = 0, pw = 0, groups = 1;
  int C = 0, H = 0, W = 0;       // per-image output shape
  Buf w, b;                      // conv [C][Cin/groups][kh][kw]; linear [C][in]
  Buf bn_g, bn_b, bn_m, bn_v;    // batchnorm
  float eps = 1e-5f;
  int copy_of = -1;
};

struct Step {
  int out = -1;                  // produced tensor (group: the root)
  std::vector<int> in;           // tensors read from outside the step
  std::vector<int> members;      // executed nodes in O order (1 for a plain op)
  bool group = false;
  std::vector<int> extra;        // further reduce outputs of a merged group (reading R37)
};

struct SkipDecision {
  int node;
  int kind;                      // 0 optimized, 1 unreducible, 2 rejected by Overhead
  std::vector<int> list;
};

struct IR {
  int batch = 0, elem = 4;       // elem = sizeof(plan dtype)
  std::vector<Node> nodes;       // by id: L (0 .. nL-1) then COPY clones
  int nL = 0, output = -1, input = 0;
  std::map<int, int64_t> orig_flops;

  std::vector<int> O;                    // optimized list (ids)
  std::vector<std::vector<int>> oin;     // inputs in O, by id
  std::map<int, std::vector<int>> groups;  // root -> members (O order)
  std::vector<Step> steps;               // schedule S
  std::vector<Step> unfused_steps;       // L as steps
  int64_t peak_fused = 0, peak_unfused = 0;
  std::vector<int64_t> live_fused, live_unfused;
  std::vector<SkipDecision> decisions;

  int64_t size(int id) const {
    const Node& n = nodes[id];
    return (int64_t)batch * n.C * n.H * n.W * elem;
  }
};

struct BuildOptions {
  int distance_threshold = 1;
  bool skip_opt = true;
  bool fusion = true;
  bool extensions = true;        // readings R34 (CP core pair), R35 (1x1 core folded into its fconv),
                                 // R36 (pool before the restore), R37 (merged fconvs), R38 (re-scheduling)
  bool cse = true;               // reading R37 (with extensions)
  int cse_policy = 0;            // 0: keep a merge iff the fused peak does not grow; 1: iff <= unfused peak
  bool reorder = true;           // reading R38 (with extensions)
  int overhead_policy = 0;       // 0 paper, 1 always, 2 never
  bool bf16 = false;
};

// Validates the user graph, expands decompositions and runs the whole rewrite.
// Returns TEMCO_OK or an error with `err` set.
temco_status build_ir(const temco_layer* layers, int n_layers, const temco_decomp* decomps, int n_decomps,
                      const temco_edge* edges, int n_edges, const temco_config& cfg, const BuildOptions& opt,
                      IR& ir, std::string& err);

int64_t node_flops(const IR& ir, int id);

}  // namespace temco
