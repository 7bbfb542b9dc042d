// tcgen05 fused-group kernels (kernels_tc.cu): lowering + launch interface.
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
  Loc r;                 // reduced input [N*H*W, R] bf16
  int32_t R, Rp;         // rank, padded to a multiple of 64 (K atoms)
  int32_t level;         // chain level this term accumulates into
  int32_t c0, C;         // restored channel range it writes (concat members)
  int64_t w;             // tc weight pool offset (elements): [C_total_rows][Rp] bf16, K-major
  alignas(64) unsigned char tmap[128];   // CUtensorMap of r (filled by tc_finalize)
  alignas(64) unsigned char wmap[128];   // CUtensorMap of the weight block
};

struct TcChainDesc {
  int32_t n_terms, n_levels;
  int32_t Ctot;          // restored width C
  int32_t Nout, Np;      // fconv outputs and padded (multiple of 16)
  int64_t npix;
  int32_t relu[kTcMaxLevels];
  int64_t bias[kTcMaxLevels];   // params offsets [C] fp32 (folded), -1 none
  int64_t F;             // tc weight pool offset: [Np][Cpad] bf16
  int32_t Cpad;          // C padded to a multiple of the chunk
  Loc y;                 // output [npix, Nout] (plan dtype)
  int64_t alg_flops, alg_bytes;
  TcTerm term[kTcMaxTerms];
  alignas(64) unsigned char fmap[128];
};

bool tc_lower_chain(const IR& ir, const Step& s, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                    std::vector<float>& params, TcChainDesc& d);
bool tc_finalize(size_t n, const std::function<TcChainDesc*(size_t)>& get, char* arena, uint16_t* tcw,
                 std::string& err);
void launch_tc_chain(const TcChainDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s);

}  // namespace temco
