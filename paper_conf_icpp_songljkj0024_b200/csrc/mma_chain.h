// Register-resident fused group kernel (kernels_mma.cu) for small restored
// widths: per warp, 16 pixels; GEMM1 (restore) accumulates in registers with
// mma.sync m16n8k16 (bf16 -> fp32), the level epilogue (bias, ReLU, running
// max for a pooled chain) runs on the accumulator fragments, and the fragments
// are re-packed in place as the A operand of GEMM2 (reduce) -- no TMEM, no
// mbarrier handoffs, so many independent warps hide the memory latency of
// these HBM-bound groups.  Same group forms as tc_chain (tc.h).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <map>
#include <vector>

#include "device.h"
#include "planner.h"

namespace temco {

constexpr int kMmaMaxTerms = 40;
constexpr int kMmaMaxLevels = 16;

struct MmaTerm {
  Loc r;              // reduced input [npix_in, R] bf16 (arena)
  int32_t R, Rp;      // rank, padded to 16
  int32_t c0, C;      // restored channel range written by this term
  int32_t level;
  int32_t w;          // element offset of Lhat [C][Rp + 8] in the smem weight blob
};

struct MmaChainDesc {
  MmaTerm term[kMmaMaxTerms];
  int32_t n_terms, n_levels;
  int32_t lvl_end[kMmaMaxLevels];
  int32_t relu[kMmaMaxLevels];
  int32_t bias[kMmaMaxLevels];      // float offset of bias [Cpad] in the blob (after the bf16 part)
  int32_t C, Cpad, CH, nchunks;     // restored width, padded to CH (64 | 128)
  int32_t Nout, Np8, f;             // F [Np8][Cpad + 8] at element offset f
  int32_t pool, pk, ps, pp, taps;
  int32_t Hin, Win, Ho, Wo;
  int64_t npix;                     // output pixels (root resolution)
  int32_t nblocks;                  // 16-pixel blocks
  Loc y;
  int64_t blob;                     // element offset of the blob in the tc weight pool
  int32_t blob_bf16;                // bf16 elements of the blob (biases follow as fp32)
  int32_t blob_bytes;
  int32_t a_stride;                 // per-warp A staging: elements per pixel row (sum of Rp + 8 per term)
  int32_t nbuf, warps;              // per-warp prefetch ring depth (units); warps per CTA
  int32_t smem_bytes;
  int64_t alg_flops, alg_bytes;
};

bool mma_lower_chain(const IR& ir, const Step& s, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                     MmaChainDesc& d);
bool mma_lean_ok(const MmaChainDesc& d);   // the lean single-term kernel applies
void launch_mma_chain(const MmaChainDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s);

}  // namespace temco
