// tcgen05 fused-group kernel, wide-group variant (kernels_tc_wide.cu): lowering + launch interface.
// Used for groups whose per-tile reduced inputs do not fit in shared memory
// (the level accumulates in TMEM over 128-channel units; see kernels_tc_wide.cu).
//
// Covers the groups whose restored tensor parses into a "level chain"
// (chain_parse.h; reading R12, P:L305-317 + P:L321-333):
//     t_1 = act_1( sum_{j in 1} Lhat_j r_j + b_1 )
//     t_l = act_l( sum_{j in l} Lhat_j r_j + b_l + t_{l-1} )      l = 2..D
// (Lhat = BN-folded lconv rows; a concat of lconvs is one level whose terms
// write disjoint channel ranges, Fig. 9a; avg-pooled linear members are
// tap-accumulate terms), optionally with one max-pooled member in the leading
// channels ("pooled chunks", evaluated per tap), followed by the root: fconv
// out = F t_D, or GAP.  bf16 ranks % 8 == 0.
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
namespace wide {

constexpr int kTcMaxTerms = 40;    // reduced inputs (lconv leaves) per group, incl. pooled-member terms
constexpr int kTcMaxLevels = 16;

struct TcTerm {
  alignas(64) unsigned char tmap[128];   // 2D map of r [npix x R], box {64, 128} (consecutive tiles)
  alignas(64) unsigned char wmap[128];   // Lhat [Cpad x Rw], box {64, Cc}
  alignas(64) unsigned char tmap4[128];  // spatial tiles: 4D map of r [N, Hin, Win, R], box {64, tw*ts, th*ts, tn}
  Loc r;                 // reduced input [N, Hin, Win, R] bf16 (arena)
  int32_t R, Rp;         // rank; padded to a multiple of the K atom
  int32_t aw;            // K atom width in elements (16 / 32 / 64 -> SW32 / SW64 / SW128 boxes)
  int32_t Rw;            // row length of the packed weights (R rounded to 8; TMA zero-fills to Rp)
  int32_t c0, C;         // restored channels this term writes (concat members)
  int32_t Hin, Win;      // resolution of r
  int32_t tk, ts, tp;    // tap-accumulate window (1 = plain term)
  int64_t w;             // tc weight pool offset (elements)
  int32_t cfirst, nhit;  // chunks [cfirst, cfirst + nhit) receive this term
  int32_t wres;          // resident mode: byte offset of [nhit][Rp/aw] boxes (Cc x aw) in the weight region
};

// Per-tile programs (host-generated, identical for every tile of a group): the
// producer and MMA roles replay flat op lists instead of re-deriving the unit /
// level / term / tap / K-atom loop nest per stage (a single issuing thread is
// latency-bound on that scalar code).
enum : uint8_t { PK_A4D = 1, PK_A2D = 2, PK_B = 4 };
struct TcProdOp {                 // one ring stage
  uint8_t kind, ts;               // PK_*; tile-base stride of a 4D A box
  uint16_t amap, bmap;            // byte offsets / 64 of the CUtensorMaps inside TcChainDesc
  int16_t ac, dx, dy;             // A coords: channel; tap offsets (4D: w0*ts+dx, h0*ts+dy)
  int16_t bx, by;                 // B coords
  uint32_t bytes;                 // expect_tx
  uint8_t n2, aw;                 // K atoms in the stage (1 or 2), atom width (elements)
  uint16_t bstep64;               // byte offset / 64 of the stage's second B atom
  uint16_t pad[4];
};
static_assert(sizeof(TcProdOp) == 32, "TcProdOp layout");
enum : uint16_t {
  MF_ACC_WAIT = 1,      // wait acc_empty[bs] first
  MF_P_WAIT = 2,        // wait p_full[unit]
  MF_OUT_WAIT = 4,      // wait out_empty
  MF_SW = 8,            // wait full[stage]
  MF_SA = 16,           // A operand = current stage slot A
  MF_SB = 32,           // B operand = current stage slot B
  MF_SD = 64,           // commit empty[stage] + advance after
  MF_ONES = 128,        // A = constant ones tile (bias MMA)
  MF_F = 256,           // fconv MMA: A = P[unit] + aoff, D = output region, N = Np
  MF_ZERO = 512,        // first MMA of the accumulator (k == 0 does not accumulate)
  MF_ACC_COMMIT = 1024, // commit acc_full[bs] after
  MF_P_COMMIT = 2048,   // commit p_empty[unit] after
  MF_OUT_COMMIT = 4096, // commit out_full after
  MF_BRES = 8192,       // B = resident weights + boff
  MF_BZERO = 16384,     // B = zero tile (with MF_ONES | MF_ZERO: zero-initialise the region)
};
struct TcMmaOp {
  uint16_t flags;
  uint8_t unit, nk;               // unit index in the tile (TMEM buffer parity) or P buffer; K=16 steps
  uint8_t la, lb;                 // K-atom widths (layouts) of A and B
  uint16_t tcol;                  // TMEM column offset inside the unit buffer
  uint32_t aoff, boff;
  uint8_t nk1;                    // two-atom stage: K=16 steps of the first atom (0: one atom)
  uint16_t a2, b2;                // descriptor deltas (>> 4) of the second atom
};
// device form: UMMA descriptors precomputed on the host relative to the
// 1024-aligned SMEM base (start-address field = offset >> 4); the issuer only
// adds (base >> 4) and, for ring operands, (stage * slot) >> 4
struct TcMmaOpD {
  uint64_t adesc, bdesc;
  uint32_t idesc, tmem;           // instruction descriptor; TMEM column (low 16 bits; unit ops: + buffer * ubuf)
                                  // bits 24-31: K=16 steps in the first atom of a two-atom stage (0: one atom)
  uint16_t flags;
  uint8_t unit, nk;
  uint16_t a2, b2;                // descriptor deltas (>> 4) of the stage's second A / B atom
};
static_assert(sizeof(TcMmaOpD) == 32, "TcMmaOpD layout");

struct TcChainDesc {
  TcTerm term[kTcMaxTerms];
  alignas(64) unsigned char fmap[128];   // F [Np x Cpad], box {64, Np}
  // level biases enter the accumulator through the tensor core: a constant
  // SMEM "ones" A tile (K columns 0, 1 = 1) times B = [b_hi, b_lo] per channel
  alignas(64) unsigned char bmap[kTcMaxLevels][128];   // [Cpad x 8] bf16, box {64, Cc}
  alignas(64) unsigned char bmapm[128];                 // pooled member bias
  int64_t boff[kTcMaxLevels];            // tc weight pool offsets of the bias matrices
  int64_t boffm;
  int64_t lbias[kTcMaxLevels], mbias;    // fp32 params offsets of the level / member biases (epilogue adds)
  int32_t n_terms, n_levels;             // outer (level) terms: [0, n_terms)
  int32_t lvl_end[kTcMaxLevels];         // terms [lvl_end[l-1], lvl_end[l]) accumulate into level l
  int32_t relu[kTcMaxLevels];
  int32_t C, Cpad, Cc, nchunks;          // restored width, padded, chunk width (64 | 128)
  int32_t Nout, Np;                      // fconv outputs, padded to a multiple of 16
  int64_t npix;                          // root-resolution pixels
  int32_t ntiles;
  int32_t rows_per_tile;                 // consecutive tiles: 128, or whole images for a GAP root
  int32_t gap, hw, ipt;                  // GAP root: pixels per image, images per tile
  int32_t nimg;
  int32_t Ho, Wo;                        // root resolution
  // spatial tiles (any tap-shifted read): tn x th x tw output pixels (<= 128)
  int32_t spatial, tw, th, tn, nwb, nhb, nnb, mused;
  // pooled member in channel chunks [0, npc): per-tap MMA regions (tpu taps per
  // unit, ntg tap groups), then pool, + post-shift (params, fp32 [npc*Cc]), act
  int32_t npc, mpool, mk, ms, mp, mtaps, mrelu, mt0, mt1, mHin, mWin;
  int32_t tpu, ntg, ubuf;                // ubuf = TMEM columns of one unit buffer
  int64_t post;                          // params offset of the post-pool shift, -1 none
  int64_t postsc;                        // params offset of the post-pool scale (SiLU members), -1 none
  int64_t F;                             // tc weight pool offset of F
  int64_t Fb;                            // unused (fconv factors carry no bias)
  Loc y;                                 // output [npix, Nout] bf16, or [N, C] for GAP
  // resident weights (every B operand fits in SMEM): loaded once per CTA, the
  // ring then carries only A tiles.  Avoids all 148 SMs re-reading the same
  // few weight lines through TMA every stage (L2 same-line contention).
  int32_t resident, wres_bytes;
  int32_t k2;                            // two K atoms per ring stage (half the stages, twice the MMAs each)
  int32_t bres[kTcMaxLevels], bresm;     // bias boxes: [nchunks] x (Cc x 16), byte offsets
  int32_t fres;                          // F boxes: [Cpad / 64] x (Np x 64)
  int64_t prog_off;                      // tc weight pool offset (elements) of [prod ops][mma ops]
  int32_t n_prod, n_mma, units;          // ops per tile; units per tile
  int32_t mma_head;                      // > 0: pipelined MMA order, unit ops = mma[0, mma_head)
  int32_t prog_smem;                     // > 0: programs copied to SMEM at kernel start (bytes reserved)
  const TcProdOp* prod;                  // device pointers (tc_finalize)
  const TcMmaOpD* mma;
  int32_t stages, slot_a, slot_b;        // smem ring depth, bytes of one A / B slot
  int32_t smem_bytes, tmem_cols;
  int64_t alg_flops, alg_bytes;          // algorithmic work (unpadded ranks), for the roofline
};

bool tc_lower_chain(const IR& ir, const Step& s, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                    std::vector<float>& params, TcChainDesc& d);
bool tc_finalize(size_t n, const std::function<TcChainDesc*(size_t)>& get, char* arena, uint16_t* tcw,
                 std::string& err);
void launch_tc_chain(const TcChainDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s);

}  // namespace wide
}  // namespace temco
