// TMA-staged reduced-rank core convolution (kernels_tile.cu): lowering + launch interface.
//
// The Tucker core K x K conv R_in -> R_out on reduced channels (Eq. (2) P:L106;
// SURVEY 8(a) row a7) and the strided 1x1 downsample cores.  HBM-bound (AI ~ 10-40 flop/B):
// a CTA stages the input footprint of an output tile with ONE 4-D TMA box (zero fill outside
// the image = the conv's zero padding), double-buffered so the next tile's footprint is in
// flight while the current one is computed; A fragments come from that footprint by ldmatrix
// (a lane per output pixel row, the tap shift is an address offset), B (weights) from SMEM,
// mma.sync m16n8k16 with fp32 accumulation, bf16 NHWC output straight from the fragments.
#pragma once

#include <cuda_runtime.h>

#include <string>
#include <vector>

#include "device.h"

namespace temco {

struct TileConvDesc {
  alignas(64) unsigned char xmap[128];   // x as (C, W, H, N) bf16, box (C, FW, FH, TN)
  Loc x, y;
  int32_t N, H, W, C, Ho, Wo, K;
  int32_t kh, kw, sh, sw, ph, pw;
  int32_t TH, TW, TN;            // output tile: rows, columns, images
  int32_t FH, FW;                // input footprint rows / columns of one image
  int32_t cw, G, RP;             // TMA view: cw pixels per inner row (cw*C*2 bytes, the swizzle span),
                                 // G inner rows per footprint row, RP = G*cw pixels per SMEM footprint row
  int32_t tiles_w, tiles_h, tiles_n, ntiles;
  int32_t pair;                  // C == 8: one k-step of 16 covers two taps
  int32_t ksc;                   // k-steps per tap (C > 8): ceil(C / 16)
  int32_t nks;                   // k-steps of the whole reduction
  int32_t swz;                   // footprint pixel row swizzle: 0 none, 1 / 2 / 3 = 32 / 64 / 128 B (TMA)
  int32_t buf_bytes;             // one footprint buffer (1024-aligned, + zeroed slack)
  int32_t box_bytes;             // TMA bytes of one footprint
  uint32_t mpx, spx, mtw, stw;   // magic multiply-high division by TH * TW and by TW
  int32_t Kp;                    // output channels padded to 16
  int32_t w_bytes;               // weights [nks][2][Kp][8] bf16 in SMEM
  int64_t wblob;                 // tc weight pool offset of the weights
  int32_t smem_bytes;
  int64_t b;                     // params offset of an fp32 bias, or -1
  int64_t alg_flops, alg_bytes;
  int32_t dbg;                   // timing experiments (TEMCO_TILE_DBG): 1 no compute, 2 no TMA
};

// w = fp32 [K][kh][kw][C]; false if the conv is outside the kernel's shapes (bf16, C % 8 == 0,
// K % 8 == 0, K <= 128, weights and two footprints within shared memory)
bool tile_conv_lower(const ConvDesc& c, const float* w, std::vector<uint16_t>& tcw, TileConvDesc& d);
bool tile_conv_finalize(TileConvDesc& d, const char* arena, std::string& err);
void launch_tile_conv(const TileConvDesc& d, const uint16_t* tcw, const RunPtrs& p, cudaStream_t s);

}  // namespace temco
