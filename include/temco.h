/*
 * temco.h -- C ABI of the B200-native TeMCO inference path.
 *
 * TeMCO (Song et al., ICPP '24; PAPER.md = /root/reference/PAPER.md, cited as
 * P:L<line>) takes "an ordered tensor node list L in SSA form" (Alg. 1 input,
 * P:L180) of a tensor-decomposed CNN and produces an optimized list whose
 * inference uses only reduced tensors:
 *   - skip connections carry the reduced tensor, the restore layers are copied
 *     before the far uses (Alg. 1/2);
 *   - lconv -> activation (-> pooling) -> fconv run as one fused kernel
 *     (P:L265-311), extended through concatenations and adds by the layer
 *     transformations of P:L321-333.
 * The three calls the north star names are temco_plan_create (layer graph,
 * decomposition ranks/factors, skip edges), temco_run (plan, input, output,
 * stream) and temco_peak_internal_bytes (Eq. (3)/(4) accounting).
 *
 * Conventions
 *  - Every function returns temco_status (0 = OK); no C++ exception crosses
 *    the ABI.  temco_last_error() gives a thread-local message for the last
 *    failure of the calling thread.
 *  - Host arrays passed to temco_plan_create are BORROWED for the duration of
 *    the call and copied; the caller may free them on return.
 *  - A plan OWNS its device weights (BN-folded, packed, plan dtype), its
 *    activation arena, TMA descriptors and (optionally) a captured CUDA graph.
 *  - A plan is bound to the CUDA device current at create time; temco_run from
 *    another current device returns TEMCO_ERR_DEVICE_MISMATCH.
 *  - temco_run is stream-ordered and asynchronous: no host synchronisation, no
 *    allocation.  A plan is NOT re-entrant (one run in flight per plan; the
 *    arena is shared).  Launch errors surface at return, asynchronous faults at
 *    the caller's next synchronisation.
 *  - There is no CPU fallback: without a device every compute call fails with
 *    TEMCO_ERR_NO_DEVICE (plans created with TEMCO_FLAG_NO_DEVICE support the
 *    host-only queries: peak bytes and describe).
 */
#ifndef TEMCO_H
#define TEMCO_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct temco_plan_s* temco_plan_t;
/* identical to cudaStream_t (struct CUstream_st*); NULL = legacy default stream */
typedef struct CUstream_st* temco_stream_t;

typedef enum {
  TEMCO_OK = 0,
  TEMCO_ERR_INVALID_ARGUMENT = 1, /* NULL pointer, bad enum, non-positive size            */
  TEMCO_ERR_INVALID_GRAPH = 2,    /* non-topological inputs, shape mismatch, skip edges   */
  TEMCO_ERR_UNSUPPORTED = 3,      /* op / rank / layout outside the supported set         */
  TEMCO_ERR_OUT_OF_MEMORY = 4,    /* device or host allocation failed                     */
  TEMCO_ERR_CUDA = 5,             /* a CUDA runtime / driver call failed                  */
  TEMCO_ERR_DEVICE_MISMATCH = 6,  /* current device differs from the plan's device        */
  TEMCO_ERR_NO_DEVICE = 7         /* compute requested on a plan without a device         */
} temco_status;

/* operators of the ORIGINAL (undecomposed) layer graph */
typedef enum {
  TEMCO_OP_INPUT = 0,          /* graph input, NHWC [batch, height, width, channels]           */
  TEMCO_OP_CONV2D = 1,         /* square kernel, stride, zero pad; groups == 1 unless undecomposed */
  TEMCO_OP_BATCHNORM = 2,      /* inference BN: gamma*(x-mean)/sqrt(var+eps)+beta              */
  TEMCO_OP_RELU = 3,
  TEMCO_OP_SILU = 4,
  TEMCO_OP_ADD = 5,            /* n-ary elementwise sum                                        */
  TEMCO_OP_CONCAT = 6,         /* channel concatenation                                        */
  TEMCO_OP_MAXPOOL = 7,        /* kernel, stride, pad (-inf padding)                           */
  TEMCO_OP_AVGPOOL = 8,        /* kernel, stride, no padding                                   */
  TEMCO_OP_GLOBAL_AVGPOOL = 9, /* mean over H, W                                               */
  TEMCO_OP_LINEAR = 10,        /* y = flatten_NCHW(x) W^T + b, W [out_channels, C*H*W]          */
  TEMCO_OP_CONV_TRANSPOSE2D = 11 /* transposed conv (UNet up-conv): square kernel,
                                  * stride, pad; H' = (H-1)*stride - 2*pad + kernel; weight
                                  * [C_in, C_out, k, k] (PyTorch ConvTranspose2d); Tucker-2 only:
                                  * first [R_in, C_in], core [R_in, R_out, k, k], last [C_out, R_out] */
} temco_op;

typedef struct {
  int32_t op;                 /* temco_op                                                        */
  int32_t n_inputs;
  const int32_t* inputs;      /* indices of EARLIER layers (SSA, execution order)               */
  int32_t out_channels;       /* conv / linear                                                   */
  int32_t kernel, stride, pad, groups;   /* conv / pool                                          */
  const float* weight;        /* conv OIHW (ignored when decomposed) / linear [out, in]; fp32    */
  const float* bias;          /* [out_channels] or NULL                                          */
  const float *bn_gamma, *bn_beta, *bn_mean, *bn_var;  /* [C] each, batchnorm only             */
  float bn_eps;
} temco_layer;

typedef enum { TEMCO_DECOMP_TUCKER2 = 1, TEMCO_DECOMP_CP = 2, TEMCO_DECOMP_TT = 3 } temco_decomp_kind;

/* decomposition of one conv layer (Eq. (2)); fp32, row-major:
 *   Tucker-2: first [rank_in, C_in] (NULL iff rank_in == C_in: no fconv),
 *             core  [rank_out, rank_in, K, K],
 *             last  [C_out, rank_out] (NULL iff rank_out == C_out: no lconv)
 *   CP      : rank_in == rank_out == R; first [R, C_in]; core = Kv [R, K];
 *             core2 = Kh [R, K]; last [C_out, R]   (fconv -> dw Kx1 -> dw 1xK -> lconv)
 *   TT      : Tensor-Train (P:L73 [28]) of W in mode order (C_in, K, K, C_out) with
 *             ranks r1 = rank_in, r2 = rank_mid, r3 = rank_out: first [r1, C_in] (NULL iff
 *             r1 == C_in), core [r2, r1, K] (a K x 1 conv, stride (s, 1), pad (p, 0)),
 *             core2 [r3, r2, K] (a 1 x K conv, stride (1, s), pad (0, p)), last [C_out, r3]
 *             (fconv -> Kx1 -> 1xK -> lconv; the lconv carries the bias)
 * Any positive rank is accepted; the tcgen05 kernels (bf16 plans) need reduced
 * ranks that are multiples of 8 (16-byte rows for TMA) and run every other
 * group on the generic SIMT kernels. */
typedef struct {
  int32_t layer;
  int32_t kind;               /* temco_decomp_kind */
  int32_t rank_in, rank_out;
  const float *first, *core, *core2, *last;
  int32_t rank_mid;           /* TT only: the rank between the two cores (ignored otherwise) */
} temco_decomp;

/* declared skip edges: must be EXACTLY the input edges (src -> dst) with
 * dst - src > 1 in layer order, else TEMCO_ERR_INVALID_GRAPH.  Alg. 1's own
 * liveness decides what is optimized; the edges are a redundancy check. */
typedef struct { int32_t src, dst; } temco_edge;

enum { TEMCO_F32 = 0, TEMCO_BF16 = 1 };

enum {
  TEMCO_FLAG_NO_DEVICE = 1 << 0,       /* plan only: no uploads, no kernels              */
  TEMCO_FLAG_NO_SKIPOPT = 1 << 1,      /* ablation: no skip connection optimization      */
  TEMCO_FLAG_NO_FUSION = 1 << 2,       /* ablation: no activation-layer fusion           */
  TEMCO_FLAG_CUDA_GRAPH = 1 << 3,      /* capture temco_run into a CUDA graph per (in,out,stream) */
  TEMCO_FLAG_SIMT_ONLY = 1 << 4,       /* never select the tcgen05 kernels               */
  TEMCO_FLAG_OVERHEAD_ALWAYS = 1 << 5, /* force Overhead() true  (tests)                 */
  TEMCO_FLAG_OVERHEAD_NEVER = 1 << 6,  /* force Overhead() false (tests)                 */
  TEMCO_FLAG_MMA_SMALL = 1 << 7,       /* run groups with C <= 256 on the mma.sync kernel */
  TEMCO_FLAG_PAPER_SCHEDULE = 1 << 9,  /* the paper's schedule exactly: without the round-2
                                          extensions R34 (CP depthwise core pair as one step),
                                          R35 (a 1x1 core folded into the fconv feeding it), R36
                                          (pool before the restore), R37 (merged fconvs) and R38
                                          (memory-optimal re-scheduling of S)                  */
  TEMCO_FLAG_MMA_CAT = 1 << 8,         /* single-level concat groups on the mma.sync concat
                                          kernel (kernels_cat.cu; measured slower than tcgen05) */
  TEMCO_FLAG_NO_CSE = 1 << 10,         /* no merged-fconv CSE (reading R37)         */
  TEMCO_FLAG_NO_RESCHEDULE = 1 << 11,  /* keep S's order (no reading R38 re-scheduling)        */
  TEMCO_FLAG_CSE_BOUND = 1 << 12       /* R37 keeps a merge iff the fused peak stays <= the
                                          unfused peak (Overhead's memory test) instead
                                          of iff it does not grow                              */
};

typedef struct {
  int32_t batch, height, width, channels;  /* input NHWC                                    */
  int32_t dtype;                           /* TEMCO_F32 | TEMCO_BF16: activations + weights */
  int32_t distance_threshold;              /* Alg. 1 DISTANCE_THRESHOLD; <= 0 -> 1 */
  int32_t flags;
} temco_config;

/* Build a plan: decomposition expansion, liveness, skip optimization
 * (Alg. 1/2), DCE, fusion grouping, BN folding, weight packing, arena
 * planning; then (unless TEMCO_FLAG_NO_DEVICE) upload to the current device. */
temco_status temco_plan_create(const temco_layer* layers, int32_t n_layers,
                               const temco_decomp* decomps, int32_t n_decomps,
                               const temco_edge* skip_edges, int32_t n_skip_edges,
                               const temco_config* cfg, temco_plan_t* out_plan);

/* Enqueue one inference on `stream`.  input: DEVICE pointer, NHWC contiguous,
 * plan dtype.  output: DEVICE pointer, fp32, [batch, classes] for a
 * linear/GAP output or NHWC [batch, H, W, C] for a feature-map output
 * (temco_output_shape). */
temco_status temco_run(temco_plan_t plan, const void* input, void* output, temco_stream_t stream);

/* Same as temco_run with HOST buffers: the input is copied host->device into a
 * plan-owned buffer, the run enqueued and the output copied device->host, all
 * on `stream`; returns after the stream has synchronised.  Pinned host memory
 * makes the copies asynchronous DMA. */
temco_status temco_run_host(temco_plan_t plan, const void* host_input, void* host_output,
                            temco_stream_t stream);

/* Asynchronous, pipelined variant of temco_run_host for a stream of batches:
 * the host->device copy of this call's input runs on a plan-owned copy stream
 * into one of two plan-owned staging buffers (alternating per call), so it
 * overlaps the previous call's compute; the run and the device->host copy of
 * the output are enqueued on `stream`.  Returns without synchronising: the
 * caller synchronises `stream` before reading host_output or reusing
 * host_input (pinned memory required for the overlap).  Consecutive calls on
 * one plan must use the same stream (the arena is shared; runs serialise). */
temco_status temco_run_host_async(temco_plan_t plan, const void* host_input, void* host_output,
                                  temco_stream_t stream);

/* Peak internal-tensor bytes (Eq. (3)/(4), reading R14): which = 0 -> the
 * fused TeMCO schedule, 1 -> the unfused decomposed list L. */
temco_status temco_peak_internal_bytes(temco_plan_t plan, int32_t which, int64_t* bytes);

/* output dims: ndim = 2 ([N, K]) or 4 (NHWC) */
temco_status temco_output_shape(temco_plan_t plan, int64_t dims[4], int32_t* ndim);

/* JSON description: schedule (steps, members, inputs, bytes), chosen kernels,
 * per-step algorithmic FLOPs / bytes, launches per run, arena size, peaks.
 * Writes at most cap bytes (NUL-terminated); *needed = full length + 1. */
temco_status temco_plan_describe(temco_plan_t plan, char* buf, size_t cap, size_t* needed);

/* Enqueue one run with a CUDA event pair around every step (profiling; no
 * CUDA graph) and, after synchronising, write per-step device milliseconds to
 * step_ms[0 .. n_steps).  n_steps must equal the schedule length. */
temco_status temco_run_profiled(temco_plan_t plan, const void* input, void* output,
                                temco_stream_t stream, float* step_ms, int32_t n_steps);

/* Verification hook (per-step parity, P:L305 / Fig. 8: every schedule step's tensor
 * of the TeMCO plan equals the same tensor of the decomposed model): enqueue
 * steps 0 .. step of one run on `stream` (no CUDA graph), synchronise, and copy
 * the output tensor of schedule step `step` (a reduced tensor in the arena,
 * NHWC in the plan dtype; or the graph output) to host_dst.  *bytes = its size;
 * host_dst = NULL only queries the size.  capacity < size ->
 * TEMCO_ERR_INVALID_ARGUMENT.  The arena is reused by later steps, so the copy
 * is taken before any later step runs.  Same device / input / output rules as
 * temco_run. */
temco_status temco_debug_step_output(temco_plan_t plan, const void* input, void* output, temco_stream_t stream,
                                     int32_t step, void* host_dst, int64_t capacity, int64_t* bytes);

/* The same for output `which` of step `step`: 0 = the step's tensor above, 1 .. = the further
 * reduce outputs of a merged group (reading R37; temco_plan_describe lists them as the
 * step's "extra"), in that order.  which out of range -> TEMCO_ERR_INVALID_ARGUMENT. */
temco_status temco_debug_step_tensor(temco_plan_t plan, const void* input, void* output, temco_stream_t stream,
                                     int32_t step, int32_t which, void* host_dst, int64_t capacity,
                                     int64_t* bytes);

temco_status temco_plan_destroy(temco_plan_t plan);
const char* temco_status_string(temco_status s);
const char* temco_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* TEMCO_H */
