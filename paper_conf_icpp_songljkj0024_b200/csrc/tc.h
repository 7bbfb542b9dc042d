// tcgen05 fused-group kernel (kernels_tc.cu): lowering + launch interface.
//
// Covers the groups whose restored tensor is a "level chain" (reading R12,
// P:L305-317 + P:L321-333):
//     t_1 = act_1( sum_{j in 1} Lhat_j r_j + b_1 )
//     t_l = act_l( sum_{j in l} Lhat_j r_j + b_l + t_{l-1} )      l = 2..D
// (Lhat = BN-folded lconv rows; a concat of lconvs is one level whose terms
// write disjoint channel ranges, Fig. 9a) followed by the root fconv
// out = F t_D.  All terms at the root resolution, bf16 ranks % 8 == 0.
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

constexpr int kTcMaxTerms = 16;    // reduced inputs (lconv leaves) per group
constexpr int kTcMaxLevels = 16;

struct TcTerm {
  alignas(64) unsigned char tmap[128];   // CUtensorMap of r  [npix x R], box {64, 128}
  alignas(64) unsigned char wmap[128];   // CUtensorMap of Lhat [Cpad x Rw], box {64, Cc}
  alignas(64) unsigned char tmap4[128];  // pooled chains: 4D map of r [N, Hin, Win, R], strided tap boxes
  Loc r;                 // reduced input [npix, R] bf16 (arena)
  int32_t R, Rp;         // rank; padded to a multiple of 64 (one 128-byte K atom)
  int32_t Rw;            // row length of the packed weights (R rounded to 8; TMA zero-fills to Rp)
  int32_t c0, C;         // restored channels this term writes (concat members)
  int64_t w;             // tc weight pool offset (elements)
};

struct TcChainDesc {
  TcTerm term[kTcMaxTerms];
  alignas(64) unsigned char fmap[128];   // CUtensorMap of F [Np x Cpad], box {64, Np}
  // level biases enter the accumulator through the tensor core: a constant
  // SMEM "ones" A tile (K columns 0, 1 = 1) times B = [b_hi, b_lo] per channel
  alignas(64) unsigned char bmap[kTcMaxLevels][128];   // CUtensorMap of [Cpad x 8] bf16, box {64, Cc}
  int64_t boff[kTcMaxLevels];            // tc weight pool offsets of the bias matrices
  int32_t n_terms, n_levels;
  int32_t lvl_end[kTcMaxLevels];         // terms [lvl_end[l-1], lvl_end[l]) accumulate into level l
  int32_t relu[kTcMaxLevels];
  int64_t bias[kTcMaxLevels];            // params offset: fp32 [Cpad] (folded BN shift + lconv biases)
  int32_t C, Cpad, Cc, nchunks;          // restored width, padded, chunk width (64 | 128)
  int32_t Nout, Np;                      // fconv outputs, padded to a multiple of 16
  int64_t npix;
  int32_t ntiles;
  int32_t rows_per_tile;                 // 128, or whole images for a GAP root
  int32_t gap, hw, ipt;                  // GAP root: pixels per image, images per tile
  int32_t nimg;
  int32_t gather;                        // A rows gathered by 4 warps (cp.async) instead of TMA
  int32_t pool, pk, ps, pp, taps;        // pooled chain: 0 none / 1 max / 2 avg, window, stride, pad
  int32_t Hin, Win, Ho, Wo;              // chain resolution, root resolution
  // pooled chains: output tiles are spatial boxes tn x th x tw (<= 128 pixels),
  // tap (dh, dw) of a term is one strided 4D TMA box (zero-filled outside)
  int32_t tw, th, tn, nwb, nhb, nnb, mused;
  int64_t F;                             // tc weight pool offset of F
  int64_t Fb;                            // params offset of the fconv bias or -1
  Loc y;                                 // output [npix, Nout] bf16
  int32_t stages, slot_b;                // smem ring depth, bytes of one B slot
  int32_t smem_bytes, tmem_cols;
  int64_t alg_flops, alg_bytes;          // algorithmic work (unpadded ranks), for the roofline
};

bool tc_lower_chain(const IR& ir, const Step& s, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                    std::vector<float>& params, TcChainDesc& d);
bool tc_finalize(size_t n, const std::function<TcChainDesc*(size_t)>& get, char* arena, uint16_t* tcw,
                 std::string& err);
void launch_tc_chain(const TcChainDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s);

}  // namespace temco
