// Launchers for the device kernels (kernels_simt.cu, kernels_tc.cu).
#pragma once

#include <cuda_runtime.h>

#include <vector>

#include <map>

#include "device.h"
#include "planner.h"

namespace temco {

void launch_conv(const ConvDesc& d, const RunPtrs& p, cudaStream_t s);
// transposed conv (UNet up-conv core): d.w = fp32 [kh*kw][K][C] (tap, out, in)
void launch_conv_transpose(const ConvDesc& d, const RunPtrs& p, cudaStream_t s);
bool conv_small_ok(const ConvDesc& d);   // small-Cin direct conv applies (stem on the image)
void launch_conv_small(const ConvDesc& d, const RunPtrs& p, cudaStream_t s);
bool conv_stem_ok(const ConvDesc& d);    // bf16 small-Cin conv on tensor cores (mma.sync, kernels_stem.cu)
void launch_conv_stem(const ConvDesc& d, const RunPtrs& p, cudaStream_t s);
// reduced-rank conv (Cin, K % 8 == 0, Cin <= 64, K <= 64) on tensor cores; w = fp32 [K][kh][kw][Cin]
bool conv_rank_mma_lower(const ConvDesc& c, const float* w, std::vector<uint16_t>& tcw, RankConvDesc& d);
void launch_conv_rank_mma(const RankConvDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s);
// single-level concat group (kernels_cat.cu); false if the group is not of that form
bool mma_cat_lower(const IR& ir, const Step& s, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                   CatDesc& d);
void launch_mma_cat(const CatDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s);
bool mma_poolcat_ok(const CatDesc& d);
bool mma_catp_ok(const CatDesc& d);      // chunk-parallel concat kernel applies (launch_mma_cat dispatches)   // restore-once 3x3/s2 max-pooled member (launch_mma_cat dispatches)
bool dwconv_vec_ok(const ConvDesc& d);   // depthwise bf16, C % 8 == 0: vectorised kernel
void launch_dwpair(const DwPairDesc& d, const RunPtrs& p, cudaStream_t s);   // CP core pair (R34)
bool dwpair_fast_ok(const DwPairDesc& d);
void launch_dwconv_vec(const ConvDesc& d, const RunPtrs& p, cudaStream_t s);
bool conv_rank_ok(const ConvDesc& d);    // reduced-rank direct conv applies (bf16, Cin, K <= 64, % 8)
void launch_conv_rank(const ConvDesc& d, const RunPtrs& p, cudaStream_t s);
void launch_ew(const EwDesc& d, const RunPtrs& p, cudaStream_t s);
void launch_linear(const LinearDesc& d, const RunPtrs& p, cudaStream_t s);
void launch_group_simt(const GroupDesc& d, const GNode* nodes, const int32_t* children, const RunPtrs& p,
                       cudaStream_t s);

}  // namespace temco
