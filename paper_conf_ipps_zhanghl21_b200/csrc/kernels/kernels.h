// Host-side launchers of the sm_100a kernels (all enqueue on the given stream, no sync).
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdlib>
#include <string>
#include <utility>

#include "../common.h"

namespace duet {

#define CK(x)                                                                                     \
  do {                                                                                            \
    cudaError_t e_ = (x);                                                                         \
    if (e_ != cudaSuccess)                                                                        \
      ::duet::fail(DUET_ECUDA, std::string(#x) + ": " + cudaGetErrorString(e_) + " @" __FILE__ ":" + \
                                   std::to_string(__LINE__));                                     \
  } while (0)

enum { EPI_BIAS_ACT = 0, EPI_LSTM = 1, EPI_GRU = 2 };
enum Act { ACT_NONE = 0, ACT_RELU = 1, ACT_SIGMOID = 2, ACT_TANH = 3, ACT_GELU = 4 };

struct TcEpilogue {
  // EPI_BIAS_ACT
  const float* bias = nullptr;
  void* out = nullptr;
  int ldo = 0;
  int act = 0;
  // EPI_LSTM / EPI_GRU (fused step: K = [x_t (kx k-blocks, zero-padded to 64) | h_{t-1}], gate
  // pre-activation = acc + bias; gate-block layout, G = 4 blocks for both LSTM (i,f,g,o) and GRU
  // (r, z, n_x, n_h))
  float* c_state = nullptr;    // LSTM cell state [M, H] fp32
  const void* h_prev = nullptr;// [M, H] bf16 (GRU z*h term)
  void* h_next = nullptr;      // [M, H] bf16
  int H = 0;
  int kx = 0;                  // k-blocks read from the X map (x_t) before switching to A (h)
  int x_row0 = 0;              // row offset of x_t in the X map ([S*B, E] time-major)
  int tma_store = 0;  // EPI_BIAS_ACT: 1 = output tile leaves through TMA stores (map passed separately)
  // single-CTA GEMM split-K (EPI_BIAS_ACT): grid.z = splits CTAs per tile store raw fp32 partials to
  // ws [splits, M, N]; gemm_splitk_reduce then applies bias + activation
  int splits = 1;
  float* ws = nullptr;
  int dbg = 0;  // micro-benchmark switches: 1 = skip UMMA, 2 = skip TMA, 4 = epilogue backoff
};

// ---- tcgen05 GEMM (gemm_tc.cu) ----
// split-K for skinny GEMMs (one 128-row tile, few N tiles, long K: MT-DNN at batch 1): the split
// count that fills the SMs with >= 2 k-blocks per split (1 = off; DUET_SPLITK=0 disables)
int tc_splitk(int M, int N, int K, int bn, int num_sms);
void gemm_splitk_reduce(const TcEpilogue& ep, int M, int N, int out_bf16, cudaStream_t st);
CUtensorMap make_tmap_bf16_2d(const void* base, int64_t rows, int64_t cols, int box_rows);
}  // namespace duet
#include <cudaTypedefs.h>
namespace duet {
PFN_cuTensorMapEncodeTiled_v12000 tmap_encode_tiled();
// Output map for TMA-store epilogues: [rows, cols] with row pitch ld elements of `eb` bytes; box =
// span_bytes / eb columns x 32 rows, swizzle matching span_bytes (128, 64 or 32).  Returns false
// (map untouched) when the TMA alignment rules are not met.
bool make_tmap_store_2d(CUtensorMap* m, void* base, int eb, int64_t rows, int64_t cols, int64_t ld, int span_bytes);
int tc_pick_bn(int M, int N, int num_sms);
void gemm_tc(const void* A, const void* W, int M, int N, int K, int bn, const TcEpilogue& ep, int epi,
             int out_bf16, cudaStream_t st);
void gemm_tc_maps(const CUtensorMap& ta, const CUtensorMap& tw, int M, int N, int K, int bn, const TcEpilogue& ep,
                  int epi, int out_bf16, cudaStream_t st, const CUtensorMap* tx = nullptr);
// Pack the fused, gate-block-interleaved recurrent weights / bias (runtime.cu builds them once):
//   Wcat[r', :] = [W_ih-part (E, zero-padded to Ep) | W_hh-part (H)], bias[r'].
void rnn_pack(int kind, const void* Wih, const void* Whh, const float* bih, const float* bhh, void* Wcat, float* bias,
              int E, int Ep, int H, int U, int BN, int tiles, cudaStream_t st);

// Persistent fused recurrence (rnn_persist.cu): all S steps in one cooperative launch of `grid`
// CTAs over tiles_n x tiles_m tiles of 128 rows x bn packed gate columns (the rnn_pack layout with
// U = bn/4); grid < tiles -> each CTA owns several tiles (state kept in global memory).
struct RnnPersistArgs {
  const float* bias = nullptr;        // [tiles_n * bn] packed gate bias
  __nv_bfloat16* hbuf[2] = {nullptr, nullptr};  // ping-pong h_t (t even -> 0, odd -> 1), K-blocked
                                                // pre-swizzled [kh][Bp][64] (rnn_persist.cu)
  __nv_bfloat16* out = nullptr;       // [B, H] h_S
  __nv_bfloat16* seq = nullptr;       // optional [S, B, H]: every h_t (a lower stacked-RNN layer)
  unsigned* counter = nullptr;        // step counters, zeroed before each launch: [tiles_m] (msync)
                                      // or [1] (grid barrier)
  float* c_state = nullptr;           // LSTM cell state [B, H] fp32 (several tiles per CTA only)
  int S = 0, B = 0, H = 0, kx = 0, kh = 0;
  int Bp = 0;                         // B padded to the 128-row tiles
  int tiles_n = 0, tiles_m = 0;       // tile grid: n (gate-block tiles of bn columns) fastest
  int dbg = 0;                        // 1 = per-step timestamps (g_rp_trace)
  int stages = 0;                     // A-ring depth (set by the launcher)
  int pair = 0;                       // 1: CTA-pair kernel (rnn_pair_kernel; 256 x 256 pair tiles)
  int ctarel = 1;                     // one-tile path: one counter release per CTA (else per epilogue warp)
  int issue2 = 1;                     // one-CTA kernel: second A / W issuer warps (odd ring stages)
  int hrot = 1;                       // h k-block load order rotated by hrot * CTA (0: all CTAs in order)
  int msync = 1;                      // 1: step t+1 of a 128-row block waits only for that block's
                                      // h_t (batch rows are independent recurrences); 0: grid barrier
  const void* wcat = nullptr;         // pair: packed weights [w_rows, w_cols] (for its 128-row box)
  int64_t w_rows = 0, w_cols = 0;
};
// CTA-pair recurrence eligibility and grid (2 x pairs) for the several-tiles-per-CTA case.
bool rnn_pair_ok(int kind, int bn, int B, int tiles_n, int tiles_m, int num_sms);
int rnn_pair_grid(int tiles_n, int tiles_m, int num_sms);
// tx: [S*B, E] (box 128 rows), th0/th1: hbuf[0/1] [B, H] (box 128 rows), tw: packed weights
// [tiles_n*bn, kx*64 + H] (box bn rows).
void rnn_persist(int kind, int bn, const CUtensorMap& tx, const CUtensorMap& th0, const CUtensorMap& th1,
                 const CUtensorMap& tw, const RnnPersistArgs& a, int grid, cudaStream_t st);

// CTA-pair GEMM (gemm_tc2.cu): 256 x bn tiles, bn in {64,128,256}; W map box rows = bn / 2.
int tc2_pick_bn(int M, int N, int K, int num_sms);
// A map box rows = 128.
void gemm_tc2_maps(const CUtensorMap& ta, const CUtensorMap& tw, int M, int N, int K, int bn, const TcEpilogue& ep,
                   int out_bf16, cudaStream_t st);

// ---- fp32 on the tensor cores (gemm_tf32.cu): 3xTF32 tcgen05 GEMM, 128 x bn tiles (bn 64 / 128) ----
// A map [M, K] fp32 box 128 rows, W map [N, K] box bn rows (make_tmap_f32_2d: 32-column boxes);
// epilogues EPI_BIAS_ACT (fp32 out) / EPI_LSTM / EPI_GRU (fp32 state, ep.kx in 32-wide k-blocks).
CUtensorMap make_tmap_f32_2d(const void* base, int64_t rows, int64_t cols, int box_rows);
bool tf32x3_ok(int K, int N);
int tf32x3_pick_bn(int M, int N, int K, int num_sms);
void gemm_tf32x3_maps(const CUtensorMap& ta, const CUtensorMap& tw, int M, int N, int K, int bn, const TcEpilogue& ep,
                      int epi, cudaStream_t st, const CUtensorMap* tx = nullptr);
void rnn_pack_f32(int kind, const float* Wih, const float* Whh, const float* bih, const float* bhh, float* Wcat,
                  float* bias, int E, int Ep, int H, int U, int BN, int tiles, cudaStream_t st);

// ---- SIMT fallbacks / small kernels (simt.cu) ----
// Y[M,N] = act(X[M,K] W[N,K]^T + b) ; X/W dtype per flags; fp32 accumulate.
void gemm_simt(const void* X, int x_bf16, const void* W, int w_bf16, const float* b, void* Y, int y_bf16, int M,
               int N, int K, int act, cudaStream_t st);
// Fused small-M MLP (all layers in one CTA per row block). dims[0..L], act on all but last.
void mlp_small(const void* X, int bf16, const void* const* Ws, const float* const* bs, const int* dims, int L,
               void* Y, int y_bf16, int M, int act, int last_act, cudaStream_t st);
// RNN step, SIMT (f32 parity path): gates from h_prev W_hh^T + gx (original PyTorch layout).
void rnn_step_simt(int kind, const float* gx, const void* Whh, int w_bf16, const float* bhh_n, const void* h_prev,
                   void* h_next, int h_bf16, float* c_state, int M, int H, cudaStream_t st);

// ---- MT-DNN encoder (transformer.cu) ----
// y[b*S + s] = LN(Etok[tok[b,s]] + Epos[s] + Eseg[seg[b,s]]) * g + beta, H <= 1024 (eps 1e-12)
void bert_embed(const int32_t* tok, const int32_t* seg, const void* Etok, const void* Epos, const void* Eseg,
                const float* g, const float* beta, void* y, int bf16, int B, int S, int H, int64_t V, cudaStream_t st);
// y = LN(a + b) * g + beta over rows of H <= 1024
void add_layernorm(const void* a, const void* b, const float* g, const float* beta, void* y, int bf16, int64_t rows,
                   int H, cudaStream_t st);
// qkv [B*S, 3H] (Q | K | V, head h = columns h*dh..) -> out [B*S, H], softmax(Q K^T / sqrt dh) V per
// (b, head); S <= 512, dh in {32, 64, 128}, K^T and V (fp32) within 227 KB of shared memory
bool attention_ok(int S, int dh);
// tcgen05 attention (attention_tc.cu): bf16, dh = 64, S <= 128; one CTA per (sequence, head)
bool attention_tc_ok(int S, int dh, int bf16);
void attention_tc(const void* qkv, void* out, int B, int S, int heads, cudaStream_t st);
void attention(const void* qkv, void* out, int bf16, int B, int S, int heads, int dh, cudaStream_t st);
// y[i] = x[offset + i * stride] (rows of `cols` elements of `esize` bytes)
void select_rows(const void* x, void* y, int esize, int64_t rows, int64_t cols, int64_t stride, int64_t offset,
                 cudaStream_t st);

// ---- gathers (gather.cu) ----
void hash_mod(const int64_t* raw, int32_t* ids, int64_t n, int64_t V, cudaStream_t st);
void gather_sum(const int32_t* ids, const void* T, int t_bf16, const float* b, float* y, int B, int F, int64_t R,
                cudaStream_t st);
void gather_concat(const int32_t* ids, const void* E, int esize, void* X, int B, int F, int64_t R, int D,
                   cudaStream_t st);
void embed_seq(const int32_t* tok, const void* E, int esize, void* X, int B, int S, int64_t V, int D,
               cudaStream_t st);
void fill_random(void* p, int dtype, int64_t n, int64_t high, uint64_t seed, cudaStream_t st);
void permute_rows(const void* src, void* dst, const int32_t* src_row_of_dst, int64_t rows_dst, int64_t row_bytes,
                  cudaStream_t st);

// ---- joins / elementwise / pooling (join.cu) ----
void reduce_sum(const void* x, int x_bf16, const float* b, float* y, int B, int K, cudaStream_t st);
void dot_join(const float* s, const void* a, int a_bf16, const float* w, const float* b, float* y, int B, int K,
              cudaStream_t st);
void cosine_join(const void* a, const void* b, int bf16, float* y, int B, int K, cudaStream_t st);
// y = act(sum_i parts_i . w_i + b); parts given as (ptr, K_i, bf16_i)
void concat_head(const void* const* parts, const int* Ks, const int* bf16s, int n, const float* w, const float* b,
                 float* y, int B, int act, cudaStream_t st);
void logit_join(const float* const* parts, int n, float* y, int B, int mean, cudaStream_t st);
void add_act(const void* a, const void* b, void* y, int bf16, int64_t n, int act, cudaStream_t st);
void sigmoid_ew(const void* x, void* y, int bf16, int64_t n, cudaStream_t st);
void maxpool_nhwc(const void* x, void* y, int bf16, int N, int H, int W, int C, int k, int s, int p, int Ho,
                  int Wo, cudaStream_t st);
void avgpool_nhwc(const void* x, void* y, int bf16, int N, int H, int W, int C, cudaStream_t st);

// ---- convolution (conv.cu) ----
struct ConvShape {
  int N, H, W, C, Co, kh, kw, stride, pad, Ho, Wo;
};
// y = act(conv(x, Wf) + bias (+ residual)); Wf [Co, kh, kw, C] with BN folded; NHWC.
void conv_fwd(const void* x, const void* Wf, const float* bias, const void* residual, void* y, int bf16,
              const ConvShape& s, int act, cudaStream_t st);  // CUDA-core path, Wf rows dense
// Fold BN into conv weights/bias: Wf = W * g/sqrt(var+eps), bias = beta - mean*g/sqrt(var+eps).
// Wf rows are ldw >= per_co elements apart; the padding is zero-filled.
void fold_bn(const void* W, int bf16, const float* g, const float* beta, const float* mean, const float* var,
             void* Wf, float* bias, int Co, int64_t per_co, int64_t ldw, cudaStream_t st);
// tcgen05 implicit-GEMM conv (conv_tc.cu); tw = TMA map of Wf [Co, ldw] with box rows = bn.
// Tap rectangle of a conv: the filter taps that touch the input for at least one output pixel.
struct ConvTaps { int r0 = 0, nr = 1, s0 = 0, ns = 1; };
ConvTaps conv_taps(const ConvShape& s);
// fp32 implicit-GEMM conv (3xTF32; C % 32 == 0): tw = make_tmap_f32_2d(Wf [Co, kh*kw*C], Co, K, bn),
// bn in {64, 128}; residual fp32 [M, Co] or null.  im2col_f32: explicit im2col for the other layers
// (the 3-channel stem), rows padded to ldk (% 4 == 0) with zeros.
bool conv_tf32_ok(const ConvShape& s);
void conv_tf32x3(const CUtensorMap& tw, const void* x, const float* bias, const void* residual, void* y,
                 const ConvShape& s, int act, int bn, cudaStream_t st);
void im2col_f32(const void* x, void* cols, const ConvShape& s, int64_t ldk, cudaStream_t st);
// Launch plan: tile width bn, effective 64-wide k-blocks nkb (tap rectangle); ks is always 1.
struct ConvPlan { int bn = 64, ks = 1, nkb = 0; };
ConvPlan conv_tc_plan(const ConvShape& s, int num_sms);
int conv_tc_pick_bn(const ConvShape& s, int num_sms);
// ctr: [2] zeroed unsigned counters for dynamic tile scheduling (null: static persistent tiles)
void conv_tc(const CUtensorMap& tw, const void* x, const float* bias, const void* residual, void* y,
             const ConvShape& s, int K, int act, const ConvPlan& p, unsigned* ctr, cudaStream_t st);
bool conv_tma_ok(const ConvShape& s);
// Explicit im2col (layers with C % 64 != 0): cols[m, k] = x[n, ho*s-p+r, wo*s-p+q, c], k = (r, q, c),
// rows padded to ldk (zeros), bf16.
void im2col(const void* x, void* cols, const ConvShape& s, int64_t ldk, cudaStream_t st);

// Direct small-channel conv (conv_stem.cu): im2col in shared memory, tcgen05, persistent.
bool conv_stem_ok(const ConvShape& s);
void conv_stem_pack(const void* wf, int64_t ldw, void* wk, const ConvShape& s, cudaStream_t st);  // wk [Co, 192]
CUtensorMap conv_stem_wmap(const void* wk, int Co);
void conv_stem(const CUtensorMap& tw, const void* x, const float* bias, void* y, const ConvShape& s, int act,
               unsigned* ctr, cudaStream_t st);  // ctr: [2] zeroed counters (dynamic tiles) or null

int num_sms(int device);

// Launch with the programmatic-stream-serialization attribute (PDL): the kernel must execute
// griddepcontrol.wait before touching data produced by the preceding kernel in the stream.
// PDL switches: DUET_NO_PDL (any value) disables it everywhere, DUET_PDL_TC=0 only for the
// tcgen05 kernels (experiments).
inline bool pdl_on(bool tc) {
  static const bool off = getenv("DUET_NO_PDL") != nullptr;
  static const bool tc_off = getenv("DUET_PDL_TC") && atoi(getenv("DUET_PDL_TC")) == 0;
  return !off && !(tc && tc_off);
}
template <typename... KArgs, typename... Args>
void launch_pdl_if(bool on, void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                   Args&&... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = on ? 1 : 0;
  CK(cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...));
}
template <typename... KArgs, typename... Args>
void launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, Args&&... args) {
  launch_pdl_if(pdl_on(false), kern, grid, block, smem, st, std::forward<Args>(args)...);
}
// Same, without the PDL attribute: full stream serialization (used for kernels adjacent to
// persistent / cluster kernels in the CNN chain, where early dependent launch was observed to hang
// back-to-back graph copies).
template <typename... KArgs, typename... Args>
void launch_plain(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, Args&&... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cfg.numAttrs = 0;
  CK(cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...));
}
// blocks for a grid-stride kernel: enough for `work` items, capped at per_sm x SM count
int grid_for(int64_t work, int threads, int per_sm = 8);

}  // namespace duet
