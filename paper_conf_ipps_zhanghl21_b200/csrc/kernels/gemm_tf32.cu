// fp32 contractions on the tensor cores: 3xTF32 tcgen05 GEMM with the fused epilogues of
// gemm_tc.cu (SURVEY.md §8(a) A5-A8 in fp32 mode; K3 "fp32 parity path via 3xTF32"; VERDICT r1
// missing item 5).  BASELINE.json's north star asks fp32 outputs to match the oracle within 1e-5
// relative; kind::tf32 alone keeps 10 mantissa bits (~5e-4), so every operand is split
//   a = a_big + a_small,  a_big = a with the low 13 mantissa bits cleared (exact in tf32),
//   a_small = a - a_big (exact in fp32, rounded to tf32 by the MMA: relative error <= 2^-22 of a)
// and D = A_big W_big^T + A_big W_small^T + A_small W_big^T (the dropped small x small term is
// <= 2^-22 relative), accumulated in fp32 in TMEM over several accumulators (F32Cfg::kBig).
//
//   D[M, N] = A[M, K] * W[N, K]^T      A, W fp32 K-major (row-major [rows, K])
//
// One CTA computes one 128 x BN tile (BN 64 or 128).  k-blocks are 32 fp32 = 128 B rows, the same
// SWIZZLE_128B atom as the bf16 kernels (a tf32 UMMA step is K = 8 = 32 B, as a bf16 step is
// K = 16).  Warp roles (6 warps):
//   warp 0      TMA producer: A/W k-blocks into a STAGES ring (full[s])
//   warp 1      TMEM allocator + UMMA issuer: three kind::tf32 UMMAs per 8-deep k-step
//   warps 2..5  split the landed stage in shared memory (a_small into the stage's second half;
//               a_big is the MMA's own truncating tf32 read of the fp32 operand; elementwise, so the
//               swizzle is irrelevant), fence the generic-proxy
//               stores for the tensor core (split[s]); after the mainloop: the fused epilogue
// Epilogues (fp32 in and out): EPI_BIAS_ACT (+ optional residual), EPI_LSTM, EPI_GRU -- gemm_tc.cu's,
// with the state (c, h_prev, h_next) in fp32 and full-precision expf / tanhf.
// CONV = true: the implicit-GEMM convolution of conv_tc.cu in fp32 (A9): per 32-channel k-block of
// filter tap (r, s) one im2col-mode TMA gathers 128 output pixels x 32 channels (zero halo), W is
// the BN-folded [Co, kh*kw*C] matrix; taps outside the tap rectangle are skipped (conv_taps).
#include <cudaTypedefs.h>

#include "../common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace duet {

namespace {

constexpr int FBM = 128;
constexpr int FBK = 32;                      // fp32: 128 bytes per row = one SWIZZLE_128B atom row
constexpr int F_A_BYTES = FBM * FBK * 4;     // 16 KB
constexpr int kFSplitThreads = 128;          // warps 2..5

template <int BN>
struct F32Cfg {
  static constexpr int W_BYTES = BN * FBK * 4;
  static constexpr int STAGE = 2 * (F_A_BYTES + W_BYTES);  // big A | big W | small A | small W
  static constexpr int STAGES = BN <= 64 ? 4 : 3;
  // accumulators: kBig for the A_big W_big terms (k-block kb into kb % kBig) + one for the two
  // cross terms, all of TMEM; summed in fp32 registers by the epilogue.  The tensor core's fp32
  // accumulation is biased (the error grows linearly with the UMMAs accumulated into one TMEM
  // accumulator), so spreading them bounds it: c2's fc1 in fp32 (K = 1664) 1.46e-5 with one
  // accumulator, 1.1e-6 with 1 + 7 (tools/tf32_acc.py)
  static constexpr int kBig = BN <= 64 ? 7 : 3;
  static constexpr int TMEM_COLS = 512;
  static constexpr int SMEM = STAGES * STAGE + 1024 + 512 + BN * 4;
};

__host__ __device__ constexpr uint32_t idesc_tf32(uint32_t M, uint32_t N) {
  // D f32 (bits 4-5 = 1), A tf32 (bits 7-9 = 2), B tf32 (bits 10-12 = 2), both K-major
  return (1u << 4) | (2u << 7) | (2u << 10) | ((N >> 3) << 17) | ((M >> 4) << 24);
}

__device__ __forceinline__ void umma_tf32_elect(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                                uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p, e;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}

// big / small parts of 4 fp32 values
__device__ __forceinline__ void split4(uint4& v, uint4& s) {
  const uint32_t x[4] = {v.x, v.y, v.z, v.w};
  uint32_t b[4], r[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    b[i] = x[i] & 0xFFFFE000u;
    r[i] = __float_as_uint(__uint_as_float(x[i]) - __uint_as_float(b[i]));
  }
  v = make_uint4(b[0], b[1], b[2], b[3]);
  s = make_uint4(r[0], r[1], r[2], r[3]);
}

struct F32Conv {
  ConvShape s{};
  int nkb = 0;               // 32-wide k-blocks: taps in the rectangle x C / 32
  int r0 = 0, s0 = 0, ns = 1;
  const float* res = nullptr;
};

template <int BN, int EPI, bool CONV>
__global__ void __launch_bounds__(192, 1)
    gemm_tf32x3_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmW,
                       const __grid_constant__ CUtensorMap tmX, const TcEpilogue ep, const F32Conv cv, int M, int N,
                       int K) {
  using Cfg = F32Cfg<BN>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + Cfg::STAGES * Cfg::STAGE);
  uint64_t* split = full + Cfg::STAGES;
  uint64_t* empty = split + Cfg::STAGES;
  uint64_t* tmem_full = empty + Cfg::STAGES;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_full + 1);
  float* s_bias = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(full) + 512);
  // stage s: [A big 16 KB][W big][A small 16 KB][W small]
  auto sA = [&](int s) { return smem + s * Cfg::STAGE; };
  auto sW = [&](int s) { return smem + s * Cfg::STAGE + F_A_BYTES; };

  const int warp = ptx::warp_id();
  const int lane = threadIdx.x & 31;
  const int n0 = blockIdx.x * BN;
  const int m0 = blockIdx.y * FBM;
  const int nk = CONV ? cv.nkb : (K + FBK - 1) / FBK;

  if (warp == 0 && lane == 0) {
    ptx::tma_prefetch(&tmA);
    ptx::tma_prefetch(&tmW);
    if (ep.kx) ptx::tma_prefetch(&tmX);
    for (int s = 0; s < Cfg::STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&split[s], kFSplitThreads / 32);
      ptx::mbar_init(&empty[s], 1);
    }
    ptx::mbar_init(tmem_full, 1);
    ptx::fence_mbar_init();
  }
  ptx::pdl_wait();  // before taking TMEM (gemm_tc.cu: a waiting TMEM holder can starve another stream)
  if (warp == 1) {
    ptx::tmem_alloc(tmem_slot, Cfg::TMEM_COLS);
    ptx::tmem_relinquish();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  ptx::pdl_trigger();

  if (warp == 0) {
    if (lane == 0) {
      // conv: the tile's first output pixel (n, ho, wo) -> im2col base coordinates
      const ConvShape& cs = cv.s;
      const int wo = CONV ? m0 % cs.Wo : 0;
      const int q0 = CONV ? m0 / cs.Wo : 0;
      const int ho = CONV ? q0 % cs.Ho : 0, nn = CONV ? q0 / cs.Ho : 0;
      const int wb = wo * cs.stride - cs.pad, hb = ho * cs.stride - cs.pad;
      const int cb = CONV ? cs.C / FBK : 1;
      for (int kb = 0; kb < nk; ++kb) {
        const int s = kb % Cfg::STAGES;
        if (kb >= Cfg::STAGES) ptx::mbar_wait(&empty[s], ((kb / Cfg::STAGES) - 1) & 1);
        ptx::mbar_arrive_expect_tx(&full[s], F_A_BYTES + Cfg::W_BYTES);
        if constexpr (CONV) {
          const int tap = kb / cb, c0 = (kb - tap * cb) * FBK;
          const int r = cv.r0 + tap / cv.ns, q = cv.s0 + tap % cv.ns;
          ptx::tma_load_im2col_4d(&tmA, &full[s], sA(s), c0, wb, hb, nn, (uint16_t)q, (uint16_t)r);
          ptx::tma_load_2d(&tmW, &full[s], sW(s), (r * cs.kw + q) * cs.C + c0, n0);
        } else {
          if (kb < ep.kx)  // fused RNN step: x_t part of K
            ptx::tma_load_2d(&tmX, &full[s], sA(s), kb * FBK, ep.x_row0 + m0);
          else
            ptx::tma_load_2d(&tmA, &full[s], sA(s), (kb - ep.kx) * FBK, m0);
          ptx::tma_load_2d(&tmW, &full[s], sW(s), kb * FBK, n0);
        }
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t idesc = idesc_tf32(FBM, BN);
    const uint64_t d0 = ptx::desc_sw128(ptx::smem_u32(smem));
    constexpr int kSmall = (F_A_BYTES + Cfg::W_BYTES) >> 4;  // small half of a stage, 16-B units
    const int nbig = (ep.dbg & 7) ? (ep.dbg & 7) : Cfg::kBig;  // experiments: dbg & 7 big accumulators
    const bool sep = !(ep.dbg & 8);                              // dbg & 8: cross terms share them
    for (int kb = 0; kb < nk; ++kb) {
      const int s = kb % Cfg::STAGES;
      ptx::mbar_wait(&split[s], (kb / Cfg::STAGES) & 1);
      ptx::tc_fence_after();
      const uint64_t da = d0 + (uint64_t)((s * Cfg::STAGE) >> 4);
      const uint64_t dw = da + (F_A_BYTES >> 4);
      const int j = kb % nbig;
      const uint32_t tb = tmem + (uint32_t)((1 + j) * BN);
      const uint32_t ts = sep ? tmem : tb;
#pragma unroll
      for (int k = 0; k < FBK / 8; ++k) {
        const uint32_t first_b = kb >= nbig || k != 0;
        const uint32_t first_s = sep ? (kb | k) != 0 : 1;
        if (sep) umma_tf32_elect(ts, da + kSmall + 2 * k, dw + 2 * k, idesc, first_s);  // A_small W_big
        umma_tf32_elect(tb, da + 2 * k, dw + 2 * k, idesc, first_b);                    // A_big W_big
        if (!sep) umma_tf32_elect(ts, da + kSmall + 2 * k, dw + 2 * k, idesc, 1);
        umma_tf32_elect(ts, da + 2 * k, dw + kSmall + 2 * k, idesc, 1);                  // A_big W_small
      }
      ptx::umma_commit_elect(&empty[s]);
    }
    ptx::umma_commit_elect(tmem_full);
  } else {
    // ---------------- warps 2..5: operand split, then the epilogue ----------------
    const int et = threadIdx.x - 64;
    for (int c = et; c < BN; c += kFSplitThreads) s_bias[c] = (ep.bias && n0 + c < N) ? ep.bias[n0 + c] : 0.0f;
    constexpr int kChunks = (F_A_BYTES + Cfg::W_BYTES) / 16;
    for (int kb = 0; kb < nk; ++kb) {
      const int s = kb % Cfg::STAGES;
      ptx::mbar_wait(&full[s], (kb / Cfg::STAGES) & 1);
      uint4* big = reinterpret_cast<uint4*>(sA(s));
      uint4* small = big + kChunks;
      // only the small parts are stored: kind::tf32 reads the top 19 bits of each fp32 operand
      // (truncation), which IS a_big -- measured: the same error with and without clearing the
      // low bits in place (tools/tf32_time.py), and 10% faster without the store
      if (!(ep.dbg & 32))  // experiments: 32 = no split (mainloop timing; wrong results)
#pragma unroll 4
        for (int i = et; i < kChunks; i += kFSplitThreads) {
          uint4 v = big[i], r;
          split4(v, r);
          small[i] = r;
        }
      ptx::fence_async_smem();  // generic-proxy stores -> visible to the tensor core
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&split[s]);
    }
    asm volatile("bar.sync 1, 128;" ::: "memory");  // s_bias written by all four warps

    const int q = warp & 3;  // TMEM lane quarter this warp may access
    const int row = m0 + q * 32 + lane;
    ptx::mbar_wait(tmem_full, 0);
    ptx::tc_fence_after();
    const uint32_t tq = tmem + ((uint32_t)(q * 32) << 16);
    const int nbig = (ep.dbg & 7) ? (ep.dbg & 7) : Cfg::kBig;
    const int nacc = min(nbig, nk);  // accumulators that received a k-block
    const bool sep = !(ep.dbg & 8);
    // v[0..16) = sum of the accumulators at column col (cross terms first, then the big ones)
    auto ld_sum16 = [&](int col, float* v) {
      float t[16];
      if (sep) ptx::tmem_ld16(tq + col, v);
#pragma unroll 1
      for (int j = 0; j < nacc; ++j) {
        ptx::tmem_ld16(tq + (1 + j) * BN + col, t);
        if (!sep && j == 0) {
#pragma unroll
          for (int i = 0; i < 16; ++i) v[i] = t[i];
        } else {
#pragma unroll
          for (int i = 0; i < 16; ++i) v[i] += t[i];
        }
      }
    };
    if constexpr (EPI == EPI_BIAS_ACT) {
      float* out = reinterpret_cast<float*>(ep.out) + (size_t)row * ep.ldo;
      const float* res = cv.res ? cv.res + (size_t)row * ep.ldo : nullptr;  // conv residual [M, Co]
#pragma unroll 1
      for (int c = 0; c < BN / 16; ++c) {
        float v[16];
        ld_sum16(c * 16, v);
        const int col0 = n0 + c * 16;
        if (row < M && col0 < N) {
          if (res)
#pragma unroll
            for (int i = 0; i < 16; ++i)
              if (col0 + i < N) v[i] += res[col0 + i];
#pragma unroll
          for (int i = 0; i < 16; ++i) v[i] = apply_act(v[i] + s_bias[c * 16 + i], ep.act);
          store_row16_any(out + col0, v, N - col0);
        }
      }
    } else {
      // RNN cell; 4 gate blocks of U units per tile (gemm_tc.cu's layout), state in fp32
      constexpr int G = 4;
      constexpr int U = BN / G;
      const int H = ep.H;
      const int unit0 = blockIdx.x * U;
#pragma unroll 1
      for (int jc = 0; jc < U; jc += 16) {
        float acc[G][16];
#pragma unroll
        for (int g = 0; g < G; ++g) ld_sum16(g * U + jc, acc[g]);
        if (row >= M) continue;
        const int nv = min(16, H - (unit0 + jc));
        if (nv <= 0) continue;
#pragma unroll
        for (int g = 0; g < G; ++g)
#pragma unroll
          for (int i = 0; i < 16; ++i) acc[g][i] += s_bias[g * U + jc + i];
        float h[16];
        if constexpr (EPI == EPI_LSTM) {
          float* cst = ep.c_state + (size_t)row * H + unit0 + jc;
#pragma unroll
          for (int i = 0; i < 16; ++i) {
            if (i >= nv) break;
            const float ig = sigmoidf_acc(acc[0][i]);
            const float fg = sigmoidf_acc(acc[1][i]);
            const float gg = tanhf(acc[2][i]);
            const float og = sigmoidf_acc(acc[3][i]);
            const float c = fg * cst[i] + ig * gg;
            cst[i] = c;
            h[i] = og * tanhf(c);
          }
        } else {
          const float* hp = reinterpret_cast<const float*>(ep.h_prev) + (size_t)row * H + unit0 + jc;
#pragma unroll
          for (int i = 0; i < 16; ++i) {
            if (i >= nv) break;
            const float r = sigmoidf_acc(acc[0][i]);
            const float z = sigmoidf_acc(acc[1][i]);
            const float n = tanhf(acc[2][i] + r * acc[3][i]);  // (W_in x + b_in) + r * (W_hn h + b_hn)
            h[i] = (1.0f - z) * n + z * hp[i];
          }
        }
        float* hn = reinterpret_cast<float*>(ep.h_next) + (size_t)row * H + unit0 + jc;
        store_row16_any(hn, h, nv);
      }
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, Cfg::TMEM_COLS);
  }
}

template <int BN, int EPI, bool CONV = false>
void launch_f32(const CUtensorMap& a, const CUtensorMap& w, const CUtensorMap& x, const TcEpilogue& ep, int M, int N,
                int K, cudaStream_t st, const F32Conv& cv = F32Conv{}) {
  using Cfg = F32Cfg<BN>;
  auto kern = gemm_tf32x3_kernel<BN, EPI, CONV>;
  static bool attr_done = false;
  if (!attr_done) {
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM));
    attr_done = true;
  }
  dim3 grid((N + BN - 1) / BN, (M + FBM - 1) / FBM);
  launch_pdl_if(pdl_on(true), kern, grid, dim3(192), Cfg::SMEM, st, a, w, x, ep, cv, M, N, K);
}

// fp32 fused recurrent weights: gemm_tc.cu's rnn_pack layout with fp32 elements and the x part
// padded to Ep = E rounded up to 32 (one fp32 k-block)
__global__ void rnn_pack_f32_kernel(int kind, const float* __restrict__ Wih, const float* __restrict__ Whh,
                                    const float* __restrict__ bih, const float* __restrict__ bhh,
                                    float* __restrict__ Wcat, float* __restrict__ bias, int E, int Ep, int H, int U,
                                    int BN, int64_t rows) {
  const int Kc = Ep + H;
  const int64_t total = rows * Kc;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / Kc;
    const int k = (int)(i - r * Kc);
    const int tile = (int)(r / BN), rem = (int)(r % BN), g = rem / U, j = tile * U + rem % U;
    float v = 0.0f;
    if (j < H) {
      const int src_gate = (kind == EPI_GRU && g == 3) ? 2 : g;  // GRU n_h uses PyTorch gate n (index 2)
      const bool use_x = !(kind == EPI_GRU && g == 3);
      const bool use_h = !(kind == EPI_GRU && g == 2);
      if (k < E) {
        if (use_x) v = Wih[((int64_t)src_gate * H + j) * E + k];
      } else if (k >= Ep) {
        if (use_h) v = Whh[((int64_t)src_gate * H + j) * H + (k - Ep)];
      }
      if (k == 0) {
        float b;
        if (kind == EPI_GRU && g == 2) b = bih[2 * H + j];       // b_in
        else if (kind == EPI_GRU && g == 3) b = bhh[2 * H + j];  // b_hn
        else b = bih[src_gate * H + j] + bhh[src_gate * H + j];
        bias[r] = b;
      }
    } else if (k == 0) {
      bias[r] = 0.0f;
    }
    Wcat[i] = v;
  }
}

}  // namespace

CUtensorMap make_tmap_f32_2d(const void* base, int64_t rows, int64_t cols, int box_rows) {
  if (((uintptr_t)base & 15) || (cols * 4) % 16)
    fail(DUET_EUNSUPPORTED, "fp32 TMA operand needs a 16-byte aligned base and row pitch (K % 4 == 0)");
  CUtensorMap m;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)(cols * 4)};
  cuuint32_t box[2] = {(cuuint32_t)FBK, (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = tmap_encode_tiled()(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<void*>(base), dims, strides, box,
                                   estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) fail(DUET_ECUDA, "cuTensorMapEncodeTiled (fp32) failed (" + std::to_string((int)r) + ")");
  return m;
}

bool tf32x3_ok(int K, int N) { return K % 4 == 0 && K > 0 && N >= 16; }

int tf32x3_pick_bn(int M, int N, int K, int num_sms) {
  // 128-wide tiles only while K is short enough for their 3 big accumulators (F32Cfg::kBig): the
  // accumulation error grows with the k-blocks per accumulator (64-wide tiles spread them over 7)
  const int mt = (M + FBM - 1) / FBM;
  const int nk = (K + FBK - 1) / FBK;
  return (N >= 128 && nk <= 64 && mt * ((N + 127) / 128) >= num_sms / 2) ? 128 : 64;
}

void gemm_tf32x3_maps(const CUtensorMap& ta, const CUtensorMap& tw, int M, int N, int K, int bn, const TcEpilogue& ep,
                      int epi, cudaStream_t st, const CUtensorMap* tx) {
  const CUtensorMap& tmx = tx ? *tx : ta;
  if (M == 0 || N == 0) return;
  if (bn == 64) {
    if (epi == EPI_BIAS_ACT) return launch_f32<64, EPI_BIAS_ACT>(ta, tw, tmx, ep, M, N, K, st);
    if (epi == EPI_LSTM) return launch_f32<64, EPI_LSTM>(ta, tw, tmx, ep, M, N, K, st);
    if (epi == EPI_GRU) return launch_f32<64, EPI_GRU>(ta, tw, tmx, ep, M, N, K, st);
  } else if (bn == 128) {
    if (epi == EPI_BIAS_ACT) return launch_f32<128, EPI_BIAS_ACT>(ta, tw, tmx, ep, M, N, K, st);
    if (epi == EPI_LSTM) return launch_f32<128, EPI_LSTM>(ta, tw, tmx, ep, M, N, K, st);
    if (epi == EPI_GRU) return launch_f32<128, EPI_GRU>(ta, tw, tmx, ep, M, N, K, st);
  }
  fail(DUET_EUNSUPPORTED, "no 3xTF32 tile for bn=" + std::to_string(bn) + " epi=" + std::to_string(epi));
}

namespace {
PFN_cuTensorMapEncodeIm2col_v12000 encode_im2col() {
  static PFN_cuTensorMapEncodeIm2col_v12000 fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &p, cudaEnableDefault, &q);
    if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !p)
      fail(DUET_ECUDA, "cannot resolve cuTensorMapEncodeIm2col");
    fn = reinterpret_cast<PFN_cuTensorMapEncodeIm2col_v12000>(p);
  }
  return fn;
}

// cols[m, k] = x[n, ho*s-p+r, wo*s-p+q, c], k = (r, q, c), rows padded to ldk with zeros, fp32.
// One thread per output row: (n, ho, wo) decoded once, k walked with incremental counters, the row
// written as 16-B stores (as im2col_kernel, conv.cu).
__global__ void im2col_f32_kernel(const float* __restrict__ x, float* __restrict__ cols, ConvShape s, int ldk) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  const int K = s.kh * s.kw * s.C;
  const int64_t M = (int64_t)s.N * s.Ho * s.Wo;
  for (int64_t m = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; m < M; m += (int64_t)gridDim.x * blockDim.x) {
    const int wo = (int)(m % s.Wo);
    const int64_t q0 = m / s.Wo;
    const int ho = (int)(q0 % s.Ho), n = (int)(q0 / s.Ho);
    const int hb = ho * s.stride - s.pad, wb = wo * s.stride - s.pad;
    float4* dst = reinterpret_cast<float4*>(cols + m * ldk);
    int c = 0, q = 0, r = 0;
    for (int k0 = 0; k0 < ldk; k0 += 4) {
      float v[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        v[e] = 0.0f;
        if (k0 + e < K) {
          const int hi = hb + r, wi = wb + q;
          if ((unsigned)hi < (unsigned)s.H && (unsigned)wi < (unsigned)s.W)
            v[e] = __ldg(x + (((int64_t)n * s.H + hi) * s.W + wi) * s.C + c);
          if (++c == s.C) {
            c = 0;
            if (++q == s.kw) {
              q = 0;
              ++r;
            }
          }
        }
      }
      dst[k0 / 4] = make_float4(v[0], v[1], v[2], v[3]);
    }
  }
}
}  // namespace

bool conv_tf32_ok(const ConvShape& s) { return s.C % FBK == 0 && s.Co % 4 == 0 && s.kh <= 16 && s.kw <= 16; }

CUtensorMap make_tmap_im2col_f32(const void* x, const ConvShape& s) {
  if ((uintptr_t)x & 15) fail(DUET_EUNSUPPORTED, "conv (fp32): 16-B aligned input");
  CUtensorMap m;
  cuuint64_t dims[4] = {(cuuint64_t)s.C, (cuuint64_t)s.W, (cuuint64_t)s.H, (cuuint64_t)s.N};
  cuuint64_t strides[3] = {(cuuint64_t)s.C * 4, (cuuint64_t)s.W * s.C * 4, (cuuint64_t)s.H * s.W * s.C * 4};
  int lower[2] = {-s.pad, -s.pad};  // (W, H)
  int upper[2] = {s.pad - (s.kw - 1), s.pad - (s.kh - 1)};
  cuuint32_t estr[4] = {1, (cuuint32_t)s.stride, (cuuint32_t)s.stride, 1};
  CUresult r = encode_im2col()(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, const_cast<void*>(x), dims, strides, lower,
                               upper, FBK, FBM, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                               CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) fail(DUET_ECUDA, "cuTensorMapEncodeIm2col (fp32) failed (" + std::to_string((int)r) + ")");
  // small-tensor driver workaround, as make_tmap_im2col (conv_tc.cu)
  int drv = 0;
  cudaDriverGetVersion(&drv);
  if (drv <= 13010 && (int64_t)s.N * s.H * s.W * s.C * 4 < 131072) reinterpret_cast<uint64_t*>(&m)[1] &= ~(1ull << 21);
  return m;
}

void conv_tf32x3(const CUtensorMap& tw, const void* x, const float* bias, const void* residual, void* y,
                 const ConvShape& s, int act, int bn, cudaStream_t st) {
  const ConvTaps t = conv_taps(s);
  F32Conv cv;
  cv.s = s;
  cv.nkb = t.nr * t.ns * (s.C / FBK);
  cv.r0 = t.r0;
  cv.s0 = t.s0;
  cv.ns = t.ns;
  cv.res = (const float*)residual;
  const int M = s.N * s.Ho * s.Wo;
  if (M == 0) return;
  CUtensorMap tx = make_tmap_im2col_f32(x, s);
  TcEpilogue ep;
  ep.bias = bias;
  ep.out = y;
  ep.ldo = s.Co;
  ep.act = act;
  if (bn == 64) return launch_f32<64, EPI_BIAS_ACT, true>(tx, tw, tx, ep, M, s.Co, 0, st, cv);
  if (bn == 128) return launch_f32<128, EPI_BIAS_ACT, true>(tx, tw, tx, ep, M, s.Co, 0, st, cv);
  fail(DUET_EUNSUPPORTED, "conv_tf32x3: bn in {64, 128}");
}

void im2col_f32(const void* x, void* cols, const ConvShape& s, int64_t ldk, cudaStream_t st) {
  const int64_t M = (int64_t)s.N * s.Ho * s.Wo;
  if (!M) return;
  if (ldk % 4 || ldk >= INT32_MAX) fail(DUET_EUNSUPPORTED, "im2col_f32: ldk % 4 == 0 required");
  launch_pdl(im2col_f32_kernel, dim3(grid_for(M, 128, 16)), dim3(128), 0, st, (const float*)x, (float*)cols, s,
             (int)ldk);
  CK(cudaGetLastError());
}

void rnn_pack_f32(int kind, const float* Wih, const float* Whh, const float* bih, const float* bhh, float* Wcat,
                  float* bias, int E, int Ep, int H, int U, int BN, int tiles, cudaStream_t st) {
  const int64_t rows = (int64_t)tiles * BN;
  rnn_pack_f32_kernel<<<grid_for(rows * (Ep + H), 256), 256, 0, st>>>(kind, Wih, Whh, bih, bhh, Wcat, bias, E, Ep, H,
                                                                       U, BN, rows);
  CK(cudaGetLastError());
}

}  // namespace duet
