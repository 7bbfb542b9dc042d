// tcgen05 GEMM with a fused bias / ReLU epilogue (kernels_gemm.cu): the classifier
// head (SURVEY 2.5 "Head": GAP -> FC, VGG / AlexNet FC stacks) and the standalone
// 1x1 convolutions of the unfused ablation plans ("Decomposed").
//
//   y[m, o] = act( sum_k x[m, k] W[o, k] + b[o] )      x [M x K] bf16 (row-major: NHWC
//   pixels or flattened features), W [O x K] bf16, fp32 accumulation in TMEM.
// Tiles of 128 rows x 256 outputs; K streamed through a TMA ring; weight-bound
// heads (few rows, huge K) split K across CTAs and reduce the fp32 partials in a
// second, deterministic pass.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <string>
#include <vector>

#include "device.h"

namespace temco {

struct GemmDesc {
  alignas(64) unsigned char amap[128];   // x [M x K] bf16, box {64, 128}
  alignas(64) unsigned char bmap[128];   // W [Opad x K] bf16, box {64, 256}
  Loc x, y;                              // y: [M x O] (fp32 or bf16 per y.dtype)
  Loc y2;                                // optional second output act(y) (a following ReLU step), where = -1: none
  int32_t M, K, O, Opad;
  int64_t w;                             // tc weight pool offset of W (elements)
  int64_t b;                             // fp32 params offset of the bias, -1 none
  int32_t relu;                          // act on y itself
  // pixel-shuffle store (a k x k / stride-k transposed conv as one GEMM, UNet up-conv core):
  // row m = (n, h, w) of an H x W input, column (i*k + j)*Co + o -> y[n, h*k+i, w*k+j, o]
  int32_t shuffle_k, sh_H, sh_W, sh_Co;
  int32_t splits, kper;                  // split-K: K atoms per split
  int32_t stages, smem_bytes;
  int64_t alg_flops, alg_bytes;
};

// w: row-major [O][K] fp32 weights (K % 8 == 0); appended bf16 to tcw (zero rows up to Opad)
bool gemm_lower(GemmDesc& d, const float* w, const std::vector<float>* bias, std::vector<uint16_t>& tcw,
                std::vector<float>& params, int64_t& ws_elems);
bool gemm_finalize(GemmDesc& d, char* arena, uint16_t* tcw, std::string& err);
void launch_gemm(const GemmDesc& d, const RunPtrs& p, float* ws, cudaStream_t s);

}  // namespace temco
