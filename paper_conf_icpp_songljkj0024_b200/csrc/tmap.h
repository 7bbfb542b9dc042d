// TMA tensor-map encoding shared by the tcgen05 / TMA kernels' finalize steps (host only).
// cuTensorMapEncodeTiled is reached through the runtime's driver entry point (the library links
// only cudart, no -lcuda).
#pragma once

#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <string>

namespace temco {

// the encoder, or nullptr with err set when the driver does not provide it
inline PFN_cuTensorMapEncodeTiled_v12000 tmap_encoder(std::string& err) {
  static PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
  if (!encode) {
    cudaDriverEntryPointQueryResult q;
    void* fn = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn) {
      err = "cuTensorMapEncodeTiled unavailable";
      return nullptr;
    }
    encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  }
  return encode;
}

// swizzle whose span is the box's inner row: 16-element K atoms -> 32 B, 32 -> 64 B, 64 -> 128 B
inline CUtensorMapSwizzle tmap_swizzle_bf16(int inner_elems) {
  return inner_elems == 64 ? CU_TENSOR_MAP_SWIZZLE_128B
         : inner_elems == 32 ? CU_TENSOR_MAP_SWIZZLE_64B
                             : CU_TENSOR_MAP_SWIZZLE_32B;
}

// 2-D bf16 tensor [outer][inner] (row-major, dense), box {box_inner, box_outer}; out-of-bounds
// elements read as zero
inline bool tmap_2d_bf16(PFN_cuTensorMapEncodeTiled_v12000 encode, void* dst, const void* base, uint64_t inner,
                         uint64_t outer, uint32_t box_inner, uint32_t box_outer, CUtensorMapSwizzle sw) {
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {inner * 2};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t es[2] = {1, 1};
  return encode(reinterpret_cast<CUtensorMap*>(dst), CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims,
                strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace temco
