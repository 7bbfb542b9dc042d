// Plain-old-data descriptors shared by the host lowering (capi.cu) and the
// device kernels (kernels_*.cu).  All activations are NHWC; every tensor is
// addressed through a Loc so that a plan can be replayed on new input /
// output pointers without touching its descriptors.
#pragma once

#include <cstdint>

namespace temco {

enum DType : int32_t { DT_F32 = 0, DT_BF16 = 1 };
enum Where : int32_t { W_ARENA = 0, W_INPUT = 1, W_OUTPUT = 2 };

struct Loc {
  int32_t where = W_ARENA;   // arena / graph input / graph output
  int32_t dtype = DT_F32;
  int64_t off = 0;           // byte offset in the arena
};

struct RunPtrs {
  char* arena;
  const void* input;
  void* output;
  const float* params;       // fp32 parameter pool (SIMT kernels)
};

#ifdef __CUDACC__
__host__ __device__ inline const void* loc_ptr(const Loc& l, const RunPtrs& p) {
  return l.where == W_INPUT ? p.input : (l.where == W_OUTPUT ? (const void*)p.output : (const void*)(p.arena + l.off));
}

// Programmatic dependent launch: kernels launched with launch_pdl may start while
// the previous kernel of the stream drains; they stage their constant operands
// (weights, fragments, barriers, TMEM) first, then pdl_wait() before the first
// read or write of any activation (it returns once the previous grid completed
// and its writes are visible), and pdl_trigger() when their CTA's work is issued.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
// early trigger right after the wait (dependents' prologues overlap this grid) -- measured:
// +7 % on ResNet-18c, -2 % on DenseNet-121 (their waiting CTAs crowd the SMs); compiled in
// only with -DTEMCO_PDL_EARLY, otherwise the trigger is the implicit one at grid completion
__device__ __forceinline__ void pdl_trigger_early() {
#ifdef TEMCO_PDL_EARLY
  pdl_trigger();
#endif
}

bool pdl_enabled();   // capi.cu: false with TEMCO_NO_PDL set

template <typename... K, typename... A>
inline cudaError_t launch_pdl(void (*kern)(K...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, A&&... args) {
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<A&&>(args)...);
}
#endif

// ---------------------------------------------------------------------------
// standalone (non-fused) operators
// ---------------------------------------------------------------------------
struct ConvDesc {             // direct NHWC convolution (fconv on full tensors, cores, depthwise, plain)
  Loc x, y;
  int32_t N, H, W, C;         // input
  int32_t Ho, Wo, K;          // output spatial, output channels
  int32_t kh, kw, sh, sw, ph, pw, groups;
  int64_t w;                  // params offset: [K][kh][kw][C/groups]
  int64_t b;                  // params offset or -1
  int64_t w2;                 // depthwise: params offset of the weights in [kh][kw][C] order, -1 none
};

// the two depthwise cores of one CP decomposition as one step (reading R34): K x 1 (vertical
// stride sv, pad pv) then 1 x K (horizontal stride sh, pad ph) on C channels; the vertical result
// never leaves registers
struct DwPairDesc {
  Loc x, y;
  int32_t N, H, W, C;         // input
  int32_t H1, Ho, Wo, K;      // rows after the vertical core, output spatial, taps
  int32_t sv, pv, sh, ph;
  int64_t wv, wh;             // params offsets: per-channel taps [C][K] of each core
  int64_t bv, bh;             // params offsets of the cores' biases, -1 none
};

struct RankConvDesc {          // reduced-rank conv on tensor cores (kernels_rank.cu), bf16
  Loc x, y;
  int32_t N, H, W, C, Ho, Wo, K;
  int32_t kh, kw, sh, sw, ph, pw;
  int32_t npix, nblocks;      // output pixels, 16-pixel blocks
  int32_t KS, NT;             // k-steps of 16 input channels, n-tiles of 8 output channels
  int32_t pair;               // Cin == 8: a k-step of 16 covers two taps
  int32_t nkc, nnc;           // 64-channel input / output chunks (wide convs)
  int32_t all_taps;           // single-k-step convs: load every tap of a block at once
  int32_t wstride;            // bf16 elements per weight row in SMEM
  int64_t wblob;              // tc weight pool offset: [tap][K][wstride] bf16
  int32_t blob_bytes;
  int64_t b;                  // params offset of an fp32 bias, or -1
  int64_t alg_flops, alg_bytes;
};

// single-level concat group on mma.sync (kernels_cat.cu)
constexpr int kCatMaxTerms = 40, kCatMaxUnits = 160, kCatMaxChunks = 32;
enum : int8_t { CU_FIRST = 1, CU_LAST = 2, CU_POOLED = 4, CU_TAP_FIRST = 8, CU_TAP_LAST = 16 };
struct CatTerm {
  Loc r;                      // reduced input [N, Hin, Win, R] bf16 (arena)
  int32_t R, ks, c0, C;       // rank, k-steps of 16, restored channel range
  int32_t Hin, Win;
  int32_t kind;               // 0 level term (tk > 1: folded avg pool), 1 pooled-member term
  int32_t tk, ts, tp;         // tap window (term or pool), stride, pad
  int32_t rs, w;              // SMEM row stride (elements), weight offset [C][rs] in the blob
};
struct CatUnit {              // one (64-channel chunk, term, tap) step of a 16-pixel block
  int16_t term, chunk;        // term -1: a chunk no term reaches
  int8_t tap, flags, nt0, nt1;   // n-tiles [nt0, nt1) of the chunk the term writes
  int32_t woff;               // weight row of n-tile nt0 in the blob (elements)
};
struct CatDesc {
  CatTerm term[kCatMaxTerms];
  CatUnit unit[kCatMaxUnits];
  int32_t n_terms, n_plain, n_units;
  int16_t chunk_u0[kCatMaxChunks + 1];   // units of chunk c: [chunk_u0[c], chunk_u0[c + 1])
  int32_t C, nchunks, Nout, NO;
  int32_t H, W, npix, nblocks;
  int32_t relu;               // level activation
  int32_t pool, pk, ps, pp, mrelu, pc0, pc1;   // pooled member: kind, window, act, chunk range
  int32_t f, fs;              // F [Nout][fs] offset (elements)
  int32_t lbias, mbias;       // fp32 offsets (floats) after the bf16 part
  int32_t blob_bf16, blob_bytes;
  int64_t blob;               // tc weight pool offset
  Loc y;                      // = ys[0]
  int32_t n_out;              // reduce outputs (a merged group, reading R37: its fconvs; mma_poolcat only)
  Loc ys[4];                  // output k: columns [ycol[k], ycol[k + 1]) of the stacked F
  int32_t ycol[5];
  int64_t alg_flops, alg_bytes;
};

enum EwKind : int32_t { EW_BN, EW_RELU, EW_SILU, EW_ADD, EW_CONCAT, EW_MAXPOOL, EW_AVGPOOL, EW_GAP };

constexpr int kMaxEwInputs = 64;
struct EwDesc {               // elementwise / pooling / concat / GAP
  int32_t kind;
  int32_t n_in;
  Loc x[kMaxEwInputs];
  int32_t xc[kMaxEwInputs];   // channels of each input (concat)
  Loc y;
  int32_t N, H, W, C;         // input spatial + output channels
  int32_t Ho, Wo;
  int32_t k, s, p;
  int64_t scale, shift;       // BN (params offsets)
};

struct LinearDesc {           // y[n, o] = b[o] + sum_k W[o, k] x[n, k], x flattened NHWC
  Loc x, y;
  int32_t N, K, O;
  int64_t w, b;               // params offsets; W already permuted to NHWC order
  int32_t relu;               // fused ReLU epilogue
};

// ---------------------------------------------------------------------------
// fused group, generic SIMT interpreter (all group shapes)
// ---------------------------------------------------------------------------
enum GOp : int32_t { G_LCONV, G_AFFINE, G_RELU, G_SILU, G_ADD, G_CONCAT, G_MAXPOOL, G_AVGPOOL, G_EXT };

struct GNode {
  int32_t op;
  int32_t C, H, W;            // output per-image shape of this node
  int32_t nin, child;         // children: children[child .. child + nin)
  int32_t k, s, p;            // pooling
  int32_t R;                  // G_LCONV: reduced channels
  Loc t;                      // G_LCONV: reduced input; G_EXT: full tensor
  int32_t tC, tH, tW;         // shape of t
  int64_t w, b;               // G_LCONV weight [C][R] / bias; G_AFFINE scale / shift
};

enum RootKind : int32_t { ROOT_FCONV, ROOT_GAP, ROOT_STORE };

struct GroupDesc {
  int32_t root;               // RootKind
  int32_t tnode;              // node index (global) whose value is the C-wide restored tensor t
  int32_t N, H, W, C;         // t's shape (root resolution)
  int32_t Nout;               // fconv output channels
  int64_t F, Fb;              // fconv weight [Nout][C] / bias (-1)
  Loc y;
};

}  // namespace temco
