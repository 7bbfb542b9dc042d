// tcgen05 implicit-GEMM convolution (kernels_conv.cu) for the standalone
// convolutions of the schedule: Tucker cores K x K on reduced channels
// (SURVEY 8(a) a7), the stem core on the 3-channel image and reduces (fconv)
// of full tensors (a8).  out[px, o] = b[o] + sum_k A[px, k] W[o, k] with
// k = ((a * kw + b) * Cin + c) (im2col order, gathered on the fly).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <map>
#include <string>
#include <vector>

#include "device.h"
#include "planner.h"

namespace temco {

struct ConvTcDesc {
  alignas(64) unsigned char wmap[128];   // CUtensorMap of W [nsl*Np x Kp], box {64, Np}
  alignas(64) unsigned char xmap[128];   // TMA mode: 4D map of x [N, H, W, Cin], box {64, tw*s, th*s, tn}
  // TMA mode (Cin % 8 == 0): output tiles are spatial boxes tn x th x tw (<= 128
  // pixels); tap (a, b) of 64-channel atom kc is one tap-shifted, strided box
  // load (hardware zero padding), K index = (tap * kpt + kc) * 64 + c
  int32_t tma, s, kpt, taps;
  int32_t tw, th, tn, nwb, nhb, nnb, mused;
  Loc x, y;
  int32_t N, H, W, Cin;
  int32_t Ho, Wo, kh, kw, sh, sw, ph, pw;
  int32_t Nout, Np;
  // output-channel slices (blockIdx.y): slice j computes channels [j*Nsl, min(Nout, (j+1)*Nsl))
  // with its own resident weight block (rows [j*Np, (j+1)*Np) of W), so wide-K cores whose
  // full weight matrix exceeds the SMEM budget still run on the tensor cores
  int32_t nsl, Nsl;
  int32_t vec;            // 1: Cin % 8 == 0 (16-byte chunks per tap); 0: element gather
  int32_t K, kchunks;     // GEMM K (kh*kw*Cin) and 16-byte chunks of it
  int32_t katoms;         // 64-wide K atoms
  int64_t npix;
  int32_t ntiles;
  int64_t w;              // tc weight pool offset [Np][katoms*64]
  int64_t b;              // params offset of the bias, -1 none
  int32_t stages, smem_bytes, tmem_cols;
  int64_t alg_flops, alg_bytes;
};

bool conv_tc_lower(const IR& ir, int out, const std::map<int, Loc>& loc, std::vector<uint16_t>& tcw,
                   std::vector<float>& params, ConvTcDesc& d);
bool conv_tc_finalize(ConvTcDesc& d, uint16_t* tcw, std::string& err);
bool conv_tc_finalize_x(ConvTcDesc& d, const void* x, std::string& err);   // TMA mode: input tensor map
void launch_conv_tc(const ConvTcDesc& d, const RunPtrs& p, cudaStream_t s);

}  // namespace temco
