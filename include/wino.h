/*
 * include/wino.h -- C ABI of libwino.so: fused batched Winograd F(2x2,3x3)
 * forward convolution for NVIDIA B200 (sm_100a).
 *
 * Method: Yan, Wang & Chu, "Optimizing Batched Winograd Convolution on GPUs"
 * (PPoPP'20).  Citations "L<n>" are lines of the paper text with the
 * section / equation they fall in; DESIGN.md lists every reading taken where
 * the text is silent or garbled.
 *
 * Conventions shared by every entry point
 * ---------------------------------------
 *  * Pointers named *_dev are caller-owned DEVICE pointers (cudaMalloc'd or
 *    equivalent) to dense, row-major fp32 tensors, 16-byte aligned; pointers
 *    named *_host are caller-owned HOST pointers (pinned memory recommended).
 *    The library never allocates, frees or retains caller memory, and keeps no
 *    state across calls other than per-device capability / attribute caches,
 *    so calls are thread-safe.
 *  * All calls are asynchronous on `stream` (a cudaStream_t; NULL = legacy
 *    default stream).  The return value reports argument validation and
 *    launch errors only; device faults surface at the caller's next
 *    synchronisation, as usual in CUDA.
 *  * Tensor layouts are the paper's (Table 4):
 *        x  (C,H,W,N)  "CHWN"     input,  N contiguous
 *        w  (C,3,3,K)  "CRSK"     filter, K contiguous
 *        u  (C,4,4,K)  "CR'S'K"   transformed filter; element (r',s') of
 *                                 G*w*G^T at [c][r'][s'][k] (reading R6)
 *        y  (K,H,W,N)  "KHWN"     output
 *  * Only pad = 1, stride = 1 are supported (ResNet 3x3 layers, Table 1):
 *    other values return WINO_ERR_UNSUPPORTED.  Any N, C, K, H, W >= 1 is
 *    accepted (L1281 states peak speed at N%32 = 0, K%64 = 0, C%8 = 0; other
 *    shapes take generic load paths, never a CPU fallback).
 *  * Errors: NULL pointer or dimension <= 0 -> WINO_ERR_INVALID_ARG;
 *    y overlapping x or u -> WINO_ERR_INVALID_ARG; a tensor of >= 2^31
 *    elements -> WINO_ERR_TOO_LARGE; a device pointer not 16-byte aligned ->
 *    WINO_ERR_MISALIGNED; current device not sm_100 -> WINO_ERR_UNSUPPORTED;
 *    a CUDA runtime failure -> WINO_ERR_CUDA (see wino_last_cuda_error()).
 *  * Output is deterministic: no atomics; split-C partial sums are reduced in
 *    a fixed order.
 */
#ifndef WINO_H_
#define WINO_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* wino_stream_t; /* identical to cudaStream_t */

typedef enum {
    WINO_OK = 0,
    WINO_ERR_INVALID_ARG = 1,
    WINO_ERR_UNSUPPORTED = 2,
    WINO_ERR_MISALIGNED = 3,
    WINO_ERR_TOO_LARGE = 4,
    WINO_ERR_CUDA = 5
} wino_status_t;

typedef enum {
    WINO_TC_TF32 = 0,   /* operands rounded to TF32 (cvt.rna), FP32 accumulate    */
    WINO_TC_3XTF32 = 1  /* big*big + big*small + small*big, ~FP32 accuracy        */
} wino_tc_mode_t;

/* Library ABI version (major*10000 + minor*100 + patch). */
int wino_version(void);

/* Human-readable name of a status code; never NULL. */
const char* wino_status_string(wino_status_t s);

/* The cudaError_t of the most recent WINO_ERR_CUDA on the calling thread (0 if none). */
int wino_last_cuda_error(void);

/*
 * Size in bytes of the transformed-filter workspace u: 16*C*K floats
 * (L993, Sec. 7.3: "16KC transformed filter data (0.25MB for Conv2, 1MB for
 * Conv3, 4MB for Conv4 and 16MB for Conv5)").  Returns 0 if C or K <= 0.
 * Pure host computation; needs no GPU.
 */
size_t wino_filter_workspace_bytes(int C, int K);

/*
 * Filter transform (FTF), Eq. 5 (L191), "separate kernel" of Sec. 3.1 (L209)
 * and Sec. 4.1 (L345):  u[c,:,:,k] = G * w[c,:,:,k] * G^T with
 * G = [[1,0,0],[1/2,1/2,1/2],[1/2,-1/2,1/2],[0,0,1]] (Eq. 3; reading R1).
 *   w_dev : (C,3,3,K) fp32, read-only
 *   u_dev : (C,4,4,K) fp32, written (wino_filter_workspace_bytes(C,K) bytes)
 * Run once per weight set; the result is consumed by wino_conv2d_f2x3_fwd*.
 */
wino_status_t wino_filter_transform(const float* w_dev, float* u_dev, int C, int K,
                                    wino_stream_t stream);

/*
 * Several filter transforms (Eq. 5) in one launch -- e.g. every layer of a network step, so the
 * per-launch latency of the small FTFs is paid once.  jobs[i]: w (C,3,3,K) -> u (C,4,4,K) as
 * wino_filter_transform; 1 <= n <= 8; the u's must not overlap each other or any w.
 * Errors as wino_filter_transform, per job.
 */
typedef struct {
    const float* w; /* (C,3,3,K) device */
    float* u;       /* (C,4,4,K) device */
    int C, K;
} wino_ftf_job_t;
wino_status_t wino_filter_transform_multi(const wino_ftf_job_t* jobs, int n, wino_stream_t stream);

/*
 * Fused forward convolution on FP32 CUDA cores (FFMA), Sec. 3-4 and
 * Algorithm 1 (L351-355): for every 4x4 input tile the input transform
 * V = B^T d B (Eq. 6), the 16 Winograd-domain batched GEMMs
 * M^(xi) = sum_c U^(xi)[c,k] V^(xi)[c,nu] (Eq. 7/9/10, L197-203, L373-395) and
 * the output transform Y = A^T M A (Eq. 8) in ONE kernel; implicit zero
 * padding (Sec. 3.5); odd H/W compute and discard the extra row/column
 * (L1155).  Computes y[k,i,j,n] = sum_{c,r,s} x[c,i+r-1,j+s-1,n] * w[c,r,s,k]
 * (Eq. 4; zero outside the image).
 *   x_dev : (C,H,W,N) fp32          u_dev : (C,4,4,K) from wino_filter_transform
 *   y_dev : (K,H,W,N) fp32, fully overwritten; must not overlap x_dev or u_dev
 *   pad, stride : must both be 1
 */
wino_status_t wino_conv2d_f2x3_fwd(const float* x_dev, const float* u_dev, float* y_dev,
                                   int N, int C, int H, int W, int K, int pad, int stride,
                                   wino_stream_t stream);

/*
 * wino_conv2d_f2x3_fwd with an explicit channel-split factor (split-C).
 * The paper's kernel gives each CTA a whole (64 filters x 32 tiles) output
 * block and all C channels (Sec. 3.3; Alg. 1); with small
 * per-rank batches (batch sharding) there are then fewer blocks
 * than SMs.  With split_c = S > 1 a thread-block cluster of S CTAs shares each
 * block, CTA r summing channels [r*C/S, (r+1)*C/S) (per 8-channel block), and
 * because the output transform is linear (Eq. 8) the S partial 2x2
 * outputs are pushed through distributed shared memory to the CTA owning the
 * filter (st.async) and summed there in a fixed order: deterministic, no
 * atomics, no workspace.  Results equal the unsplit kernel's up to FP32
 * summation order (bit-identical on small-integer inputs).
 *   split_c : 0 = the library's choice (what wino_conv2d_f2x3_fwd does),
 *             1, 2, 4 or 8 = forced; anything else -> WINO_ERR_INVALID_ARG.
 *             Honoured by the warp-specialised kernel (N % 32 == 0 or
 *             N in {4, 8, 16}, K % 4 == 0); other shapes ignore it.
 * Other arguments, layouts and errors as wino_conv2d_f2x3_fwd.
 */
wino_status_t wino_conv2d_f2x3_fwd_split(const float* x_dev, const float* u_dev, float* y_dev,
                                         int N, int C, int H, int W, int K, int pad, int stride,
                                         int split_c, wino_stream_t stream);

/*
 * NCHW front end (NEXT row N2; Sec. 8.4: "The implementation in this
 * work can be ported to NCHW layout with little effort ... The offsets of global
 * and shared memory accesses need to be recomputed, while all other
 * optimizations can be adopted").  Same computation as wino_conv2d_f2x3_fwd
 * (Eq. 4 via Eq. 5-8), PyTorch's default layouts:
 *   wino_filter_transform_kcrs : w_kcrs_dev (K,C,3,3) fp32 (torch conv weight)
 *                                -> u_dev (C,4,4,K), identical to
 *                                wino_filter_transform of the CRSK permutation.
 *   wino_conv2d_f2x3_fwd_nchw  : x_nchw_dev (N,C,H,W), u_dev (C,4,4,K)
 *                                -> y_nkhw_dev (N,K,H,W), fully overwritten.
 * The input tiles are gathered with per-CTA offset tables (4 B cp.async, zero
 * fill = padding) and the tiles of one image are the fastest-varying part of
 * nu; the FFMA micro-kernel and output transform are the FP32 kernel's.
 * Arguments, alignment, aliasing and errors as wino_conv2d_f2x3_fwd.
 */
wino_status_t wino_filter_transform_kcrs(const float* w_kcrs_dev, float* u_dev, int C, int K,
                                         wino_stream_t stream);
wino_status_t wino_conv2d_f2x3_fwd_nchw(const float* x_nchw_dev, const float* u_dev, float* y_nkhw_dev,
                                        int N, int C, int H, int W, int K, int pad, int stride,
                                        wino_stream_t stream);

/*
 * NEXT row N3: the NON-fused F(2x2,3x3) forward convolution -- the strategy the
 * paper's fused kernel is measured against (Sec. 9: "store intermediate
 * results in global memory ... can utilize optimized batched matrix
 * multiplication routines. However, it needs significant amount of global
 * memory as workspace and data loading can be the new bottleneck"; Sec. 7.3
 * obs. 4-6 L1159-1241; the Sec. 8.1 break-even model L1245-1269).  Four
 * launches on `stream`, all of them this library's kernels:
 *   1. u (C,4,4,K) -> Ug[16 P][K][Cp4] in ws_dev: the GEMM operand layout (channel c
 *      contiguous, row pitch Cp4 = 4*ceil(C/4)), rounded to TF32 (RNA, reading R8),
 *   2. ITF kernel: x (C,H,W,N) -> V[16 P][NV][Cp4] in ws_dev (Eq. 6), rounded likewise,
 *   3. 16 batched GEMMs M[xi][k][nu] = sum_c V[xi][nu][c] Ug[xi][k][c] (Eq. 7) on the
 *      tcgen05 tensor cores (kind::tf32, FP32 accumulation in TMEM) -> M[16][K][NV] in ws_dev,
 *   4. OTF kernel: M -> y (K,H,W,N) (Eq. 8).
 * This entry point is the FP32-accuracy variant: 3xTF32 with P = 2 planes per operand (big =
 * rna(v), small = rna(v - big); D += Vb Ub + Vb Us + Vs Ub), within the FP32 bar (<= 1e-4 of
 * max|y|) and exact on small integers.  NV = N*ceil(H/2)*ceil(W/2).  ws_dev: caller-owned
 * device workspace of at least wino_nonfused_workspace_bytes(N,C,H,W,K) = 128*NV*Cp4 +
 * 128*K*Cp4 + 64*K*NV bytes (each part rounded up to 256 B), 16-byte aligned, must not overlap
 * x, u or y; clobbered.  Other arguments, layouts and errors as wino_conv2d_f2x3_fwd;
 * ws_bytes too small -> WINO_ERR_INVALID_ARG; 32*Cp4*NV or 16*K*NV >= 2^31 ->
 * WINO_ERR_TOO_LARGE.  wino_nonfused_launches() = 4 (kernels per call).
 */
/*
 * NCHW with a device workspace: x is transposed to the paper's CHWN layout in the
 * workspace, the fused FP32 convolution runs on it (warp-specialised / stream-K plans,
 * as wino_conv2d_f2x3_fwd_ws), and y is transposed from KHWN to NKHW.  Two HBM-bound
 * transposes (8 B per element each) buy the CHWN kernel's TMA path; faster than the
 * strided gather of wino_conv2d_f2x3_fwd_nchw on every BASELINE layer.
 *   ws_dev / ws_bytes : >= wino_nchw_workspace_bytes(N,C,H,W,K) bytes = |x| + |y| (fp32,
 *                       each rounded up to 256 B) + wino_conv_workspace_bytes; 16-byte
 *                       aligned, not overlapping x, u or y; zero-filled before its first
 *                       use (the stream-K flags, as wino_conv2d_f2x3_fwd_ws), clobbered.
 * Arguments and errors as wino_conv2d_f2x3_fwd_nchw, plus WINO_ERR_INVALID_ARG for a
 * NULL or short workspace.
 */
size_t wino_nchw_workspace_bytes(int N, int C, int H, int W, int K);
wino_status_t wino_conv2d_f2x3_fwd_nchw_ws(const float* x_nchw_dev, const float* u_dev, float* y_nkhw_dev,
                                           int N, int C, int H, int W, int K, int pad, int stride,
                                           void* ws_dev, size_t ws_bytes, wino_stream_t stream);
size_t wino_nonfused_workspace_bytes(int N, int C, int H, int W, int K);
wino_status_t wino_conv2d_f2x3_fwd_nonfused(const float* x_dev, const float* u_dev, float* y_dev,
                                            int N, int C, int H, int W, int K, int pad, int stride,
                                            void* ws_dev, size_t ws_bytes, wino_stream_t stream);
int wino_nonfused_launches(void);
/* The same in plain TF32 (P = 1 plane per operand, half the V / Ug workspace traffic;
 * accuracy as the TF32 fused kernel, <= 5e-3 of max|y|; exact on small integers).  Uses a
 * prefix of the same workspace. */
wino_status_t wino_conv2d_f2x3_fwd_nonfused_tf32(const float* x_dev, const float* u_dev, float* y_dev,
                                                 int N, int C, int H, int W, int K, int pad, int stride,
                                                 void* ws_dev, size_t ws_bytes, wino_stream_t stream);

/*
 * The fused FP32 convolution with a caller-provided device workspace, which lets the
 * library run the warp-specialised kernel in stream-K mode: the tiles x channel-block
 * iteration space is cut into one equal contiguous range per SM (Alg. 1's loop over C,
 * L351-355, split across CTAs at range boundaries), partial tiles are written to the
 * workspace and a second small kernel adds each cut tile's partial outputs (Eq. 8 is
 * linear) in a fixed order -- deterministic, no atomics.  It removes the wave
 * quantisation of tiles over SMs (e.g. 392 tiles on 148 SMs) and keeps small per-rank
 * batches (batch sharding) on every SM.
 *   ws_dev / ws_bytes : >= wino_conv_workspace_bytes(N,C,H,W,K) bytes (SM count x 64 KiB of
 *                       partial tiles + one 4-byte arrival counter per SM, rounded to 256 B;
 *                       the current device's SM count, 148 when no device is current),
 *                       16-byte aligned, not overlapping x, u or y; may be NULL / 0 when
 *                       sk = 1.  The stream-K plan reduces the tiles cut between CTAs inside
 *                       the kernel: every piece of a cut tile leaves its partial outputs in the
 *                       workspace and counts itself on a GPU-scope arrival counter; the last
 *                       piece to arrive sums them (in CTA order) and stores y.  The counters
 *                       must be ZERO before the first use of a workspace (zero-fill it, e.g.
 *                       cudaMemset); every call leaves them zero again, so one initialisation
 *                       serves any number of calls on one stream (concurrent calls must not
 *                       share a workspace).
 *   sk                : 0 = the planner's choice (stream-K where its estimate beats the
 *                       regular / split-C plans and the workspace suffices), 1 = never,
 *                       2 = always when the warp-specialised kernel applies
 *                       (N % 32 == 0 or N in {4, 8, 16}, K % 4 == 0; else the regular
 *                       plan).  sk = 2 with a short workspace -> WINO_ERR_INVALID_ARG.
 * Arguments and errors otherwise as wino_conv2d_f2x3_fwd.
 */
size_t wino_conv_workspace_bytes(int N, int C, int H, int W, int K);
wino_status_t wino_conv2d_f2x3_fwd_ws(const float* x_dev, const float* u_dev, float* y_dev,
                                      int N, int C, int H, int W, int K, int pad, int stride,
                                      int sk, void* ws_dev, size_t ws_bytes, wino_stream_t stream);

/*
 * Several INDEPENDENT layers (a network step's convolutions, each with its own x, u, y and
 * shape; pad 1, stride 1) through as few launches as pay (Sec. 3-4 method per layer, Eq. 4-8;
 * the batching across layers is this library's, not the paper's).  Layers that the
 * warp-specialised FP32 kernel takes (N % 32 == 0 or N in {4, 8, 16}; K % 4 == 0) and that have
 * fewer than 64 output tiles (64 filters x 32 positions) per SM share ONE persistent launch per
 * group of up to 4: the (tile, channel block) units of the group are concatenated and cut into one
 * contiguous range per SM, balanced on a work model (unit cost per x box mode, one output
 * transform per tile), so the group pays one pipeline fill and one tail instead of one per layer,
 * and each CTA has at most two cut tiles (reduced inside the kernel as in
 * wino_conv2d_f2x3_fwd_ws).  Any other layer runs alone through wino_conv2d_f2x3_fwd_ws's
 * planner (sk = 0).  Same arithmetic per output as wino_conv2d_f2x3_fwd_ws (equal up to FP32
 * summation order of cut tiles; bit-identical on small-integer inputs).  Batch shards with N = 4
 * or 8 do not load x through 32/N TMA boxes of N-float rows: a separate input-transform kernel writes
 * their V = B^T d B (Eq. 6, same arithmetic as the fused ITF, so bit-identical) into the workspace
 * and the fused kernel loads V tiles directly ("vmode").  Launches go to `stream`: first the
 * input transforms (they read x only), then -- when `u_ready` is not NULL -- a wait on that
 * cudaEvent_t (e.g. recorded after the filter transform on another stream, so both overlap),
 * then the convolutions.
 *   jobs[i]          : device pointers and shape of layer i; y of a job must not overlap any
 *                      job's x, u or y; 1 <= n.
 *   ws_dev / ws_bytes: >= wino_conv_multi_workspace_bytes(jobs, n) (the stream-K slots and
 *                      counters of wino_conv_workspace_bytes, plus 16 x C x NV floats per vmode
 *                      layer), 16-byte aligned, not overlapping any tensor, ZERO-FILLED before
 *                      its first use (the arrival counters; every call leaves them zero).
 *   u_ready          : NULL, or a cudaEvent_t the convolutions wait for (not the input transforms).
 * Errors as wino_conv2d_f2x3_fwd_ws, per job, all checked before anything is launched;
 * n <= 0 or jobs == NULL -> WINO_ERR_INVALID_ARG.
 * wino_conv_multi_launches: kernel launches one such call makes (host only; -1 on bad input).
 */
typedef struct {
    const float* x; /* (C,H,W,N) device */
    const float* u; /* (C,4,4,K) device (wino_filter_transform) */
    float* y;       /* (K,H,W,N) device */
    int N, C, H, W, K;
} wino_conv_job_t;
size_t wino_conv_multi_workspace_bytes(const wino_conv_job_t* jobs, int n);
wino_status_t wino_conv2d_f2x3_fwd_multi(const wino_conv_job_t* jobs, int n, void* ws_dev, size_t ws_bytes,
                                         void* u_ready, wino_stream_t stream);
int wino_conv_multi_launches(const wino_conv_job_t* jobs, int n);

/*
 * Tensor-core variant (a5' of SURVEY 8(a)): the Winograd-domain GEMM (Eq. 7)
 * on the 5th-generation tensor cores (tcgen05.mma kind::tf32, accumulators in
 * TMEM).  The paper has no tensor-core path ("the data layout needs a
 * redesign", Sec. 8.3); this is the B200 redesign named in
 * BASELINE.json's north_star.  mode selects TF32 (operands rounded to TF32,
 * ~5e-4 relative) or 3xTF32 (big*big + big*small + small*big, ~FP32 accuracy).
 *
 * Its filter transform writes the transformed filter straight into the tensor
 * core's operand layout (TF32-rounded; 3xTF32 adds the residual plane):
 *   u_tc : wino_filter_workspace_bytes_tc(C,K,mode) bytes, opaque layout
 *          [ceil(C/8)][ceil(K/128)][16][planes][128 x 8 K-major tile], zero padded.
 * Arguments and errors otherwise as the FP32 entry points, plus
 * WINO_ERR_INVALID_ARG for an unknown mode.
 */
size_t wino_filter_workspace_bytes_tc(int C, int K, wino_tc_mode_t mode);
wino_status_t wino_filter_transform_tc(const float* w_dev, float* u_tc_dev, int C, int K,
                                       wino_tc_mode_t mode, wino_stream_t stream);
wino_status_t wino_conv2d_f2x3_fwd_tc(const float* x_dev, const float* u_tc_dev, float* y_dev,
                                      int N, int C, int H, int W, int K, int pad, int stride,
                                      wino_tc_mode_t mode, wino_stream_t stream);
/* The same with a caller workspace that enables a stream-K plan for tile-starved shapes (as
 * wino_conv2d_f2x3_fwd_half_ws; only the TMA x paths, N % 32 == 0 or N in {4, 8, 16}):
 *   ws_dev / ws_bytes : >= wino_tc_workspace_bytes(N,C,H,W,K) (SMs x 128 KiB), 16-byte aligned,
 *                       not overlapping x, u_tc or y; may be NULL / 0 when sk = 1.
 *   sk                : 0 = planner's choice, 1 = never, 2 = always (short workspace or a
 *                       gather-path N -> WINO_ERR_INVALID_ARG). */
size_t wino_tc_workspace_bytes(int N, int C, int H, int W, int K);
wino_status_t wino_conv2d_f2x3_fwd_tc_ws(const float* x_dev, const float* u_tc_dev, float* y_dev,
                                         int N, int C, int H, int W, int K, int pad, int stride,
                                         wino_tc_mode_t mode, int sk, void* ws_dev, size_t ws_bytes,
                                         wino_stream_t stream);

/*
 * NEXT row N4: 16-bit version on the tensor cores.  The paper:
 * "The implementation can be ported to the fp16 version by increasing bn to 64.
 * To further increase the throughput with newly introduced tensor core, the data
 * layout needs a redesign" (Sec. 8.3).  Here x, w and y are stored in the
 * 16-bit type `type` (IEEE fp16 or bfloat16, raw 2-byte elements, same layouts as
 * the FP32 calls: x (C,H,W,N), w (C,3,3,K), y (K,H,W,N)); the transforms and the
 * accumulation over C run in FP32 (tcgen05.mma kind::f16, FP32 accumulators in
 * TMEM); U, V and y are rounded to `type` with round-to-nearest-even (DESIGN.md
 * reading R18).  Accuracy: max|y - y_ref| / max|y_ref| <= 5e-3 (fp16) and 3e-2
 * (bf16) against Eq. 4 of the 16-bit inputs; bit-exact (y == round(y_ref)) on
 * small-integer inputs.
 *   u_h : wino_filter_workspace_bytes_half(C,K) bytes, opaque layout
 *         [ceil(C/16)][ceil(K/MM)][16][MM x 16 K-major tile], zero padded, with the
 *         tile height MM = 64 when K <= 64, else 128.
 * Any N, C, K, H, W >= 1; N % 32 == 0 or N in {8, 16} take TMA loads.  Errors as
 * the FP32 calls, plus WINO_ERR_INVALID_ARG for an unknown `type`.
 */
typedef enum {
    WINO_HALF_FP16 = 0, /* IEEE 754 binary16 */
    WINO_HALF_BF16 = 1  /* bfloat16          */
} wino_half_t;
size_t wino_filter_workspace_bytes_half(int C, int K);
wino_status_t wino_filter_transform_half(const void* w_dev, void* u_h_dev, int C, int K, wino_half_t type,
                                         wino_stream_t stream);
wino_status_t wino_conv2d_f2x3_fwd_half(const void* x_dev, const void* u_h_dev, void* y_dev,
                                        int N, int C, int H, int W, int K, int pad, int stride,
                                        wino_half_t type, wino_stream_t stream);
/* The same with a caller workspace that enables a stream-K plan (as wino_conv2d_f2x3_fwd_ws:
 * equal (tile, channel block) ranges on every SM; pieces of cut tiles leave FP32 partial
 * outputs in the workspace, a fixup kernel adds them in CTA order and rounds once):
 *   ws_dev / ws_bytes : >= wino_half_workspace_bytes(N,C,H,W,K) (SMs x 128 KiB), 16-byte
 *                       aligned, not overlapping x, u or y; may be NULL / 0 when sk = 1.
 *   sk                : 0 = planner's choice, 1 = never, 2 = always (a short workspace ->
 *                       WINO_ERR_INVALID_ARG). */
size_t wino_half_workspace_bytes(int N, int C, int H, int W, int K);
wino_status_t wino_conv2d_f2x3_fwd_half_ws(const void* x_dev, const void* u_h_dev, void* y_dev,
                                           int N, int C, int H, int W, int K, int pad, int stride,
                                           wino_half_t type, int sk, void* ws_dev, size_t ws_bytes,
                                           wino_stream_t stream);

/*
 * End-to-end call on HOST buffers: copies w_host and x_host to the device,
 * runs the filter transform and the fused FP32 convolution, and copies y back
 * to y_host, all enqueued on `stream` (so the call returns before the copies
 * finish; synchronise the stream before reading y_host).
 *   x_host (C,H,W,N), w_host (C,3,3,K) : read;  y_host (K,H,W,N) : written
 *   ws_dev / ws_bytes : caller-owned device workspace of at least
 *                       wino_host_workspace_bytes(N,C,H,W,K) bytes
 * Host buffers should be page-locked for the copies to be asynchronous.
 */
size_t wino_host_workspace_bytes(int N, int C, int H, int W, int K);
wino_status_t wino_conv2d_f2x3_fwd_host(const float* x_host, const float* w_host, float* y_host,
                                        int N, int C, int H, int W, int K, int pad, int stride,
                                        void* ws_dev, size_t ws_bytes, wino_stream_t stream);

/*
 * NEXT row N1: fused Winograd F(4x4,3x3), FP32 FFMA.  The paper
 * restricts itself to F(2x2,3x3) (L117) and anticipates a well-optimised fused
 * F(4x4,3x3) (Sec. 8.1).  Lavin-Gray matrices (6x6 windows at stride 4,
 * 36 Winograd elements, 4x4 outputs per tile); same computation (Eq. 4).
 *   u4 : (C,6,6,K) = G4 w G4^T, element (r',s') at [c][r'][s'][k]
 *        (36*C*K floats, wino_filter_workspace_bytes_f4)
 * Any N, C, K, H, W >= 1 (L1281): N % 16 == 0 and K % 4 == 0 take TMA boxes, other
 * shapes a cp.async gather of the same stages (generic path, same arithmetic).
 * Arguments and errors as the F(2x2) calls.
 */
size_t wino_filter_workspace_bytes_f4(int C, int K);
wino_status_t wino_filter_transform_f4(const float* w_dev, float* u4_dev, int C, int K, wino_stream_t stream);
wino_status_t wino_conv2d_f4x3_fwd(const float* x_dev, const float* u4_dev, float* y_dev,
                                   int N, int C, int H, int W, int K, int pad, int stride,
                                   wino_stream_t stream);
/* The same with a caller workspace that enables a stream-K plan (the scheme of
 * wino_conv2d_f2x3_fwd_ws: equal (tile, 4-channel block) ranges per SM, pieces of cut tiles
 * leave their 16 partial outputs per (k, nu) in the workspace, a fixup kernel adds them in CTA
 * order):  ws >= wino_f4_workspace_bytes(N,C,H,W,K) (SMs x 128 KiB), 16-byte aligned, not
 * overlapping x, u4 or y; sk 0 = planner's choice, 1 = never, 2 = always. */
size_t wino_f4_workspace_bytes(int N, int C, int H, int W, int K);
wino_status_t wino_conv2d_f4x3_fwd_ws(const float* x_dev, const float* u4_dev, float* y_dev,
                                      int N, int C, int H, int W, int K, int pad, int stride,
                                      int sk, void* ws_dev, size_t ws_bytes, wino_stream_t stream);

/*
 * Multi-layer end-to-end call on HOST buffers with copy/compute overlap: for
 * each layer the weights and input are copied in on a library-owned copy-in
 * stream, the FTF + fused FP32 convolution run on `stream`, and the output is
 * copied back on a library-owned copy-out stream in K-slices (or batch slices
 * when K < 128), so H2D of layer l+1, compute of layer l and D2H of layer l-1
 * proceed concurrently over PCIe.  `stream` is joined before returning-order
 * completion: work enqueued on `stream` after this call sees all outputs.
 * The two helper streams are created once per device (cached, like the
 * attribute caches); every event a call needs is created before anything is
 * queued, and released at the end of the call.  Errors: argument / shape errors
 * return before any work is queued; an error after work was queued (a failed
 * copy or launch) still makes `stream` wait for everything already queued on
 * the helper streams, so the caller may free or reuse its host buffers once
 * `stream` has drained.
 *   layers[i] : host pointers and shape of layer i (pad 1, stride 1)
 *   ws_dev    : device workspace of >= wino_host_multi_workspace_bytes() bytes
 */
typedef struct {
    const float* x_host; /* (C,H,W,N) */
    const float* w_host; /* (C,3,3,K) */
    float* y_host;       /* (K,H,W,N) */
    int N, C, H, W, K;
} wino_host_layer_t;
size_t wino_host_multi_workspace_bytes(const wino_host_layer_t* layers, int n_layers);
wino_status_t wino_conv2d_f2x3_fwd_host_multi(const wino_host_layer_t* layers, int n_layers, void* ws_dev,
                                              size_t ws_bytes, wino_stream_t stream);

/*
 * Launch plan the library would use for a shape (host only, needs no GPU);
 * used by tests and by bench.py to count launches and report tiling.
 */
typedef struct {
    int variant;        /* 0 = FP32 FFMA fused kernel, 1 / 2 = tcgen05 TF32 / 3xTF32, */
                        /* 3 = tcgen05 kind::f16 (FP16 / BF16, NEXT row N4),          */
                        /* 4 = FP32 with a stream-K workspace (wino_conv2d_f2x3_fwd_ws, sk = 0) */
                        /* 5 = FP16 / BF16 with a stream-K workspace (..._half_ws, sk = 0)     */
                        /* 6 / 7 = TF32 / 3xTF32 with a stream-K workspace (..._tc_ws, sk = 0) */
    int bk, bn, bc;     /* filters, tiles and channels per CTA step (Sec. 3.3)      */
    int load_x, load_u; /* how x / u reach shared memory: 0 = cp.async 4 B,         */
                        /* 1 = cp.async 16 B, 2 = TMA tiled box (cp.async.bulk.tensor) */
    int split_c;        /* channel split factor (1 = none)                          */
    int64_t ctas;       /* CTAs of the main kernel                                  */
    int threads;        /* threads per CTA                                          */
    int smem_bytes;     /* dynamic shared memory per CTA                            */
    int launches;       /* kernels launched by one wino_conv2d_f2x3_fwd* call       */
    int stream_k;       /* 1: stream-K plan (variants 4 - 7)                        */
} wino_plan_t;

wino_status_t wino_plan(int N, int C, int H, int W, int K, int variant, wino_plan_t* plan);

#ifdef __cplusplus
}
#endif
#endif /* WINO_H_ */
