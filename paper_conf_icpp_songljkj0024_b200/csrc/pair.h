// tcgen05 CTA-pair fused restore-chain kernel (kernels_pair.cu): lowering + launch interface.
//
// One fused group (Listing 1, P:L321-333 add/concat merges; reading R12)
// whose restored tensor parses into a level chain (chain_parse.h)
//     t_1 = act_1( sum_{j in 1} Lhat_j r_j + b_1 )
//     t_l = act_l( sum_{j in l} Lhat_j r_j + b_l + t_{l-1} )      l = 2..D
//     out = F t_D                                                  (the next fconv)
// with every term spanning the whole restored width C (the ResNet residual
// chains: skip restores and the block's own lconv, P:L263 / Fig. 8) and the
// fconv as root.  A 2-CTA cluster runs cta_group::2 MMAs with M = 256 pixels
// (128 per CTA): each SM stages its own pixels' reduced inputs and HALF of each
// 128-channel weight unit.  Every level's product a_l = sum_j Lhat_j r_j goes to
// a FRESH TMEM accumulator (B rotating buffers), and the epilogue keeps t in
// registers (t = act(t + a_l + b_l)), so no MMA ever waits for an epilogue
// result: the tensor pipe only waits for a free buffer, B-1 levels later.
// After the last level the epilogue writes bf16 P = t_D into shared memory and
// out += P F_u^T accumulates over the 128-channel units in its own TMEM region.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <functional>
#include <map>
#include <string>
#include <vector>

#include "device.h"
#include "planner.h"

namespace temco {
namespace pair {

constexpr int kPairMaxTerms = 32;
constexpr int kPairMaxUnitPairs = 16;    // C <= 4096
constexpr int kPairMaxLevels = 16;
constexpr int kPairMaxAtoms = 256;      // K atoms of all unit pairs' programs
constexpr int kPairMaxActGroups = 256;  // (level, 32-channel group) activation codes
constexpr int kPairWu = 128;           // restored channels per unit (MMA N of the restore GEMM)
constexpr int kPairMaxOuts = 4;        // reduce outputs of a merged group (reading R37)

struct PairTerm {
  alignas(64) unsigned char amap[128];   // r_j [npix x R] bf16, box {aw, 128}
  alignas(64) unsigned char wmap[128];   // Lhat_j [Cpad x Rw] bf16, box {aw, 64} (this CTA's half of a unit)
  Loc r;                                 // reduced input (arena)
  int32_t R, aw, natoms, Rw;             // rank, K atom width (16/32/64), atoms, packed row length
  int64_t w;                             // tc weight pool offset (elements)
};

struct PairDesc {
  PairTerm term[kPairMaxTerms];
  alignas(64) unsigned char fmap[128];   // F [Np x Cpad] bf16, box {64, Np/2}
  alignas(64) unsigned char bmap[128];   // bias-MMA groups: [n_levels*Cpad x 16] bf16 (hi, lo), box {16, 64}
  int32_t n_terms, n_levels;
  uint32_t prog[kPairMaxAtoms][2];       // atom programs: term | aw << 8 | K16 steps << 16 | flags << 24 | level << 28; x
  int32_t n_prog;                        // atoms of all programs
  int16_t pstart[kPairMaxUnitPairs];     // unit pair pp's program: atoms [pstart[pp], next 'last' flag]; a
                                         // concat term only appears in the pairs whose channels it covers
  int32_t lvl_end[kPairMaxLevels];       // terms [lvl_end[l-1], lvl_end[l]) belong to level l
  int32_t act[kPairMaxLevels];           // 0 none, 1 ReLU, 2 SiLU
  int32_t mixed_act, ngroups;            // per-channel-group activations (activated concat members)
  uint8_t actg[kPairMaxActGroups];       // [level][32-channel group] activation code when mixed_act
  int64_t lbias;                         // params offset: fp32 [n_levels][Cpad] level biases
  int32_t bias_mma;                      // level biases added by a K=16 MMA (ones x [hi, lo]) instead of the epilogue
  int64_t bmat;                          // tc weight pool offset of the bias-MMA matrix
  int32_t C, Cpad, nunits;               // restored width, padded to 128, 128-channel units
  int32_t nbuf;                          // rotating level accumulators (TMEM columns [0, 128 nbuf))
  int32_t Nout, Np;                      // fconv outputs, padded to 16
  int64_t npix;                          // pixels (rows of r_j and y)
  int32_t ntiles;                        // 256-pixel pair tiles
  int32_t n_out;                         // reduce outputs (1; a merged group, reading R37: its fconvs)
  Loc ys[kPairMaxOuts];                  // output k: [npix x (ycol[k+1] - ycol[k])] bf16 (arena) = out
  int32_t ycol[kPairMaxOuts + 1];        //   columns [ycol[k], ycol[k+1]) of the concatenated F
  int64_t F;                             // tc weight pool offset of F
  int32_t stages, slot, smem_bytes, bias_bytes;   // ring depth, stage bytes
  int32_t sa, sb;                        // ring stage: r atom bytes, one unit's Lhat-half bytes (then bias atoms)
  // resident-weight mode (every Lhat / bias / F atom of this CTA's halves fits in SMEM next
  // to a deep ring): the weights are loaded once per CTA and the ring carries only the
  // reduced-input atoms r_j, so several tiles' loads are in flight (small-C groups)
  int32_t resident, res_bytes, res_tx;   // resident region bytes, TMA bytes per CTA
  int32_t bsz, fsz;                      // resident Lhat atom slot (64 x awmax bf16), F atom (Np/2 x 64 bf16)
  int32_t res_c, res_f;                  // offsets of the bias-MMA and F atoms in the resident region
  int32_t silu;                          // some level is SiLU: SILU kernel instantiation
  int32_t flag;                          // the previous unit pair's fconv is issued after this level of the
                                         // next pair (and the out tile drained after it): the epilogue's P
                                         // writes have that many levels of slack before the issuer waits
  int64_t alg_flops, alg_bytes;          // algorithmic work (unpadded ranks), for the roofline
};

bool pair_lower_chain(const IR& ir, const Step& s, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                      std::vector<float>& params, PairDesc& d);
bool pair_finalize(size_t n, const std::function<PairDesc*(size_t)>& get, char* arena, uint16_t* tcw,
                   std::string& err);
void launch_pair_chain(const PairDesc& d, const RunPtrs& p, cudaStream_t s);

}  // namespace pair
}  // namespace temco
