// tcgen05 + TMA GEMM tile for sm_100a with fused epilogues.
//
//   D[M, N] = A[M, K] * W[N, K]^T      A, W bf16 K-major (row-major [rows, K]); fp32 accumulate
//
// One CTA computes one 128 x BN tile.  Warp roles (6 warps):
//   warp 0      TMA producer: A/W k-blocks of 64 (128-B rows, SWIZZLE_128B) into a STAGES ring
//   warp 1      TMEM allocator + single-thread tcgen05.mma issuer (UMMA 128 x BN x 16)
//   warps 2..5  epilogue: tcgen05.ld TMEM -> registers -> fused epilogue -> global
// Epilogues:
//   EPI_BIAS_ACT  out = act(acc + bias[n])                      (MLP / projections, A5-A6)
//   EPI_LSTM      fused step: a = [x_t | h_{t-1}] [W_ih | W_hh]^T + b; c = f*c + i*g; h = o*tanh(c)
//                 (A6+A7, PyTorch gate order i,f,g,o)
//   EPI_GRU       fused step with 4 gate blocks r, z, n_x = W_in x + b_in, n_h = W_hn h + b_hn:
//                 n = tanh(n_x + r*n_h); h = (1-z) n + z h (A6+A8)
// For the RNN epilogues the weight rows are gate-block interleaved per tile: tile columns
// [g*u, (g+1)*u) hold gate block g of hidden units [tile*u, (tile+1)*u), u = BN / 4, so one thread
// owns every gate of its units, and the input projection is part of the K loop (no G_x buffer;
// DESIGN.md "Data layout").
#include <cudaTypedefs.h>

#include <cstdio>

#include "../common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace duet {

namespace {

constexpr int BM = 128;
constexpr int BK = 64;  // bf16: 128 bytes per row = one SWIZZLE_128B atom row
constexpr int A_STAGE_BYTES = BM * BK * 2;

template <int BN>
struct TileCfg {
  static constexpr int B_STAGE_BYTES = BN * BK * 2;
  static constexpr int STAGES = BN <= 64 ? 8 : (BN <= 128 ? 6 : 4);
  static constexpr int TMEM_COLS = BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : 256;
  static constexpr int SMEM = STAGES * (A_STAGE_BYTES + B_STAGE_BYTES) + 1024 + 256 + BN * 4;
};

// Round 2: W k-blocks on their own issuing warp (warp 6; one thread's copies complete in issue order,
// DESIGN.md "Persistent recurrence"); ep.dbg & 64: one producer (comparisons)
template <int BN, int EPI, typename OutT>
__global__ void __launch_bounds__(224, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmW,
                   const __grid_constant__ CUtensorMap tmX, const TcEpilogue ep, int M, int N, int K) {
  using Cfg = TileCfg<BN>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + Cfg::STAGES * A_STAGE_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(sB + Cfg::STAGES * Cfg::B_STAGE_BYTES);
  uint64_t* empty = full + Cfg::STAGES;
  uint64_t* tmem_full = empty + Cfg::STAGES;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_full + 1);
  float* s_bias = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(full) + 256);

  const int warp = ptx::warp_id();
  const int lane = threadIdx.x & 31;
  const int n0 = blockIdx.x * BN;
  const int m0 = blockIdx.y * BM;
  // split-K (EPI_BIAS_ACT with ep.splits > 1): CTA z accumulates k-blocks [kb0, kb1) and stores the
  // raw fp32 partial tile to ep.ws[z]; gemm_splitk_reduce adds the splits in order (deterministic)
  const int nk_all = (K + BK - 1) / BK;
  const int per = ep.splits > 1 ? (nk_all + ep.splits - 1) / ep.splits : nk_all;
  const int kb0 = ep.splits > 1 ? (int)blockIdx.z * per : 0;
  const int nk = ep.splits > 1 ? min(nk_all, kb0 + per) - kb0 : nk_all;

  if (warp == 0 && lane == 0) {
    ptx::tma_prefetch(&tmA);
    ptx::tma_prefetch(&tmW);
    if (ep.kx) ptx::tma_prefetch(&tmX);
    for (int s = 0; s < Cfg::STAGES; ++s) {
      ptx::mbar_init(&full[s], (ep.dbg & 66) ? 1 : 2);  // A producer (+ W issuer)
      ptx::mbar_init(&empty[s], 1);
    }
    ptx::mbar_init(tmem_full, 1);
    ptx::fence_mbar_init();
  }
  const bool wsplit = !(ep.dbg & 66);
  // wait for the previous kernel BEFORE taking tensor memory: a PDL-dependent CTA that holds TMEM
  // while it waits can starve a co-resident kernel of another stream (observed as a hang with
  // two slots)
  ptx::pdl_wait();
  if (warp == 1) {
    ptx::tmem_alloc(tmem_slot, Cfg::TMEM_COLS);
    ptx::tmem_relinquish();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;     // A / gx / c_state / h_prev come from the previous kernel in the stream
  ptx::pdl_trigger();

  if (warp == 0) {
    if (lane == 0) {
      for (int i = 0; i < nk; ++i) {
        const int s = i % Cfg::STAGES;
        const int kb = kb0 + i;
        if (i >= Cfg::STAGES) ptx::mbar_wait(&empty[s], ((i / Cfg::STAGES) - 1) & 1);
        if (ep.dbg & 2) {
          ptx::mbar_arrive(&full[s]);
        } else {
          ptx::mbar_arrive_expect_tx(&full[s], A_STAGE_BYTES + (wsplit ? 0 : Cfg::B_STAGE_BYTES));
          if (kb < ep.kx)  // fused RNN step: x_t part of K
            ptx::tma_load_2d(&tmX, &full[s], sA + s * A_STAGE_BYTES, kb * BK, ep.x_row0 + m0);
          else
            ptx::tma_load_2d(&tmA, &full[s], sA + s * A_STAGE_BYTES, (kb - ep.kx) * BK, m0);
          if (!wsplit) ptx::tma_load_2d(&tmW, &full[s], sB + s * Cfg::B_STAGE_BYTES, kb * BK, n0);
        }
      }
    }
  } else if (warp == 6) {
    // W issuer (weights: graph parameters, independent of the previous kernel)
    if (lane == 0 && wsplit) {
      for (int i = 0; i < nk; ++i) {
        const int s = i % Cfg::STAGES;
        const int kb = kb0 + i;
        if (i >= Cfg::STAGES) ptx::mbar_wait(&empty[s], ((i / Cfg::STAGES) - 1) & 1);
        ptx::mbar_arrive_expect_tx(&full[s], Cfg::B_STAGE_BYTES);
        ptx::tma_load_2d(&tmW, &full[s], sB + s * Cfg::B_STAGE_BYTES, kb * BK, n0);
      }
    }
  } else if (warp == 1) {
    // the whole warp walks the k loop (uniform descriptors); elect.sync issues each UMMA
    constexpr uint32_t idesc = ptx::idesc_bf16(BM, BN);
    const uint64_t da0 = ptx::desc_sw128(ptx::smem_u32(sA));
    const uint64_t db0 = ptx::desc_sw128(ptx::smem_u32(sB));
    for (int kb = 0; kb < nk; ++kb) {  // kb counts this CTA's k-blocks (split-K: from kb0)
      const int s = kb % Cfg::STAGES;
      ptx::mbar_wait(&full[s], (kb / Cfg::STAGES) & 1);
      ptx::tc_fence_after();
      // descriptor start address is bits [0, 14) in 16-byte units: offsets add directly
      const uint64_t da = da0 + (uint64_t)((s * A_STAGE_BYTES) >> 4);
      const uint64_t db = db0 + (uint64_t)((s * Cfg::B_STAGE_BYTES) >> 4);
#pragma unroll
      for (int k = 0; k < BK / 16; ++k) {
        if (ep.dbg & 1) break;
        ptx::umma_bf16_elect(tmem, da + 2 * k, db + 2 * k, idesc, (kb | k) != 0);
      }
      ptx::umma_commit_elect(&empty[s]);
    }
    ptx::umma_commit_elect(tmem_full);
  } else {
    // ---------------- epilogue warps 2..5 ----------------
    const int q = warp & 3;  // TMEM lane quarter this warp may access
    const int row = m0 + q * 32 + lane;
    {  // bias tile -> smem (both epilogue kinds)
      const int et = threadIdx.x - 64;
      for (int c = et; c < BN; c += 128) s_bias[c] = (ep.bias && n0 + c < N) ? ep.bias[n0 + c] : 0.0f;
      asm volatile("bar.sync 1, 128;" ::: "memory");
    }
    if (ep.dbg & 4) {
      const uint32_t a = ptx::smem_u32(tmem_full);
      while (!ptx::mbar_try_wait(a, 0)) __nanosleep(256);
    } else {
      ptx::mbar_wait(tmem_full, 0);
    }
    ptx::tc_fence_after();
    const uint32_t tq = tmem + ((uint32_t)(q * 32) << 16);
    if constexpr (EPI == EPI_BIAS_ACT) {
      OutT* out = reinterpret_cast<OutT*>(ep.out) + (size_t)row * ep.ldo;
      const int act = ep.act;
      if (ep.splits > 1) {  // raw fp32 partial -> ws[z][row][col]
        float* wsr = ep.ws + ((size_t)blockIdx.z * M + row) * N;
#pragma unroll 1
        for (int c = 0; c < BN / 16; ++c) {
          float v[16];
          ptx::tmem_ld16(tq + c * 16, v);
          const int col0 = n0 + c * 16;
          if (row < M && col0 < N) store_row16_any(wsr + col0, v, N - col0);
        }
      } else
#pragma unroll 1
      for (int c = 0; c < BN / 16; ++c) {
        float v[16];
        ptx::tmem_ld16(tq + c * 16, v);
        const int col0 = n0 + c * 16;
        if (row < M && col0 < N) {
          bias_act<16>(v, s_bias + c * 16, act);
          store_row16_any(out + col0, v, N - col0);
        }
      }
    } else {
      // RNN cell epilogue; 4 gate blocks of U units per tile: block g at columns [g*U, (g+1)*U)
      constexpr int G = 4;
      constexpr int U = BN / G;
      const int H = ep.H;
      const int unit0 = blockIdx.x * U;
#pragma unroll 1
      for (int jc = 0; jc < U; jc += 16) {
        float acc[G][16];
#pragma unroll
        for (int g = 0; g < G; ++g) ptx::tmem_ld16(tq + g * U + jc, acc[g]);
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
          float cv[16];
          if (nv == 16) {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              const float4 t = reinterpret_cast<const float4*>(cst)[i];
              cv[4 * i] = t.x;
              cv[4 * i + 1] = t.y;
              cv[4 * i + 2] = t.z;
              cv[4 * i + 3] = t.w;
            }
          } else {
#pragma unroll
            for (int i = 0; i < 16; ++i) cv[i] = i < nv ? cst[i] : 0.0f;
          }
#pragma unroll
          for (int i = 0; i < 16; ++i) {
            const float ig = sigmoidf_acc(acc[0][i]);
            const float fg = sigmoidf_acc(acc[1][i]);
            const float gg = tanhf(acc[2][i]);
            const float og = sigmoidf_acc(acc[3][i]);
            cv[i] = fg * cv[i] + ig * gg;
            h[i] = og * tanhf(cv[i]);
          }
          if (nv == 16) {
#pragma unroll
            for (int i = 0; i < 4; ++i)
              reinterpret_cast<float4*>(cst)[i] = make_float4(cv[4 * i], cv[4 * i + 1], cv[4 * i + 2], cv[4 * i + 3]);
          } else {
#pragma unroll
            for (int i = 0; i < 16; ++i)
              if (i < nv) cst[i] = cv[i];
          }
        } else {
          const __nv_bfloat16* hp = reinterpret_cast<const __nv_bfloat16*>(ep.h_prev) + (size_t)row * H + unit0 + jc;
          float hpv[16];
          if (nv == 16) {
            const uint4 p0 = *reinterpret_cast<const uint4*>(hp);
            const uint4 p1 = *reinterpret_cast<const uint4*>(hp + 8);
            const __nv_bfloat16* b0 = reinterpret_cast<const __nv_bfloat16*>(&p0);
            const __nv_bfloat16* b1 = reinterpret_cast<const __nv_bfloat16*>(&p1);
#pragma unroll
            for (int i = 0; i < 8; ++i) {
              hpv[i] = __bfloat162float(b0[i]);
              hpv[8 + i] = __bfloat162float(b1[i]);
            }
          } else {
#pragma unroll
            for (int i = 0; i < 16; ++i) hpv[i] = i < nv ? __bfloat162float(hp[i]) : 0.0f;
          }
#pragma unroll
          for (int i = 0; i < 16; ++i) {
            const float r = sigmoidf_acc(acc[0][i]);
            const float z = sigmoidf_acc(acc[1][i]);
            const float n = tanhf(acc[2][i] + r * acc[3][i]);  // (W_in x + b_in) + r * (W_hn h + b_hn)
            h[i] = (1.0f - z) * n + z * hpv[i];
          }
        }
        __nv_bfloat16* hn = reinterpret_cast<__nv_bfloat16*>(ep.h_next) + (size_t)row * H + unit0 + jc;
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

// out[m, n] = act(sum_z ws[z, m, n] + bias[n]), z in order (deterministic split-K)
template <typename OutT>
__global__ void gemm_splitk_reduce_kernel(const float* __restrict__ ws, const float* __restrict__ bias, OutT* out,
                                          int M, int N, int ldo, int splits, int act) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  const int64_t total = (int64_t)M * N;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int m = (int)(e / N), n = (int)(e - (int64_t)m * N);
    float v = 0.0f;
    for (int z = 0; z < splits; ++z) v += __ldcg(ws + (size_t)z * total + e);
    out[(size_t)m * ldo + n] = from_f<OutT>(apply_act(v + (bias ? bias[n] : 0.0f), act));
  }
}

PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
    if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !p)
      fail(DUET_ECUDA, "cannot resolve cuTensorMapEncodeTiled");
    fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  }
  return fn;
}

template <int BN, int EPI, typename OutT>
void launch_tc(const CUtensorMap& a, const CUtensorMap& w, const CUtensorMap& x, const TcEpilogue& ep, int M, int N,
               int K, cudaStream_t st) {
  using Cfg = TileCfg<BN>;
  auto kern = gemm_tc_kernel<BN, EPI, OutT>;
  static bool attr_done = false;  // per instantiation; device attribute applies process-wide
  if (!attr_done) {
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM));
    attr_done = true;
  }
  dim3 grid((N + BN - 1) / BN, (M + BM - 1) / BM, ep.splits > 1 ? ep.splits : 1);
  launch_pdl_if(pdl_on(true), kern, grid, dim3(224), Cfg::SMEM, st, a, w, x, ep, M, N, K);
}

// Fused recurrent weights: row r' = tile*BN + g*U + j' <-> (gate block g, unit j = tile*U + j');
// columns [0, E) from W_ih, [E, Ep) zero, [Ep, Ep+H) from W_hh.  LSTM blocks i,f,g,o take PyTorch
// gate g of both matrices; GRU blocks r, z take gate 0/1 of both, n_x = (W_in | 0), n_h = (0 | W_hn).
__global__ void rnn_pack_kernel(int kind, const __nv_bfloat16* __restrict__ Wih, const __nv_bfloat16* __restrict__ Whh,
                                const float* __restrict__ bih, const float* __restrict__ bhh,
                                __nv_bfloat16* __restrict__ Wcat, float* __restrict__ bias, int E, int Ep, int H,
                                int U, int BN, int64_t rows) {
  const int Kc = Ep + H;
  const int64_t total = rows * Kc;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / Kc;
    const int k = (int)(i - r * Kc);
    const int tile = (int)(r / BN), rem = (int)(r % BN), g = rem / U, j = tile * U + rem % U;
    float v = 0.0f;
    if (j < H) {
      const int src_gate = (kind == 2 && g == 3) ? 2 : g;  // GRU n_h uses PyTorch gate n (index 2)
      const bool use_x = !(kind == 2 && g == 3);
      const bool use_h = !(kind == 2 && g == 2);
      if (k < E) {
        if (use_x) v = __bfloat162float(Wih[((int64_t)src_gate * H + j) * E + k]);
      } else if (k >= Ep) {
        if (use_h) v = __bfloat162float(Whh[((int64_t)src_gate * H + j) * H + (k - Ep)]);
      }
      if (k == 0) {
        float b;
        if (kind == 2 && g == 2) b = bih[2 * H + j];        // b_in
        else if (kind == 2 && g == 3) b = bhh[2 * H + j];   // b_hn
        else b = bih[src_gate * H + j] + bhh[src_gate * H + j];
        bias[r] = b;
      }
    } else if (k == 0) {
      bias[r] = 0.0f;
    }
    Wcat[i] = __float2bfloat16_rn(v);
  }
}

}  // namespace

void rnn_pack(int kind, const void* Wih, const void* Whh, const float* bih, const float* bhh, void* Wcat, float* bias,
              int E, int Ep, int H, int U, int BN, int tiles, cudaStream_t st) {
  const int64_t rows = (int64_t)tiles * BN;
  rnn_pack_kernel<<<grid_for(rows * (Ep + H), 256), 256, 0, st>>>(
      kind, (const __nv_bfloat16*)Wih, (const __nv_bfloat16*)Whh, bih, bhh, (__nv_bfloat16*)Wcat, bias, E, Ep, H, U,
      BN, rows);
  CK(cudaGetLastError());
}

CUtensorMap make_tmap_bf16_2d(const void* base, int64_t rows, int64_t cols, int box_rows) {
  if (((uintptr_t)base & 15) || (cols * 2) % 16)
    fail(DUET_EUNSUPPORTED, "TMA operand needs 16-byte aligned base and row pitch (K % 8 == 0)");
  CUtensorMap m;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)(cols * 2)};
  cuuint32_t box[2] = {(cuuint32_t)BK, (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = get_encode()(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box,
                            estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) fail(DUET_ECUDA, "cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ")");
  return m;
}

PFN_cuTensorMapEncodeTiled_v12000 tmap_encode_tiled() { return get_encode(); }

bool make_tmap_store_2d(CUtensorMap* m, void* base, int eb, int64_t rows, int64_t cols, int64_t ld, int span_bytes) {
  if (((uintptr_t)base & 15) || (ld * eb) % 16 || cols * eb < span_bytes || rows < 32) return false;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)(ld * eb)};
  cuuint32_t box[2] = {(cuuint32_t)(span_bytes / eb), 32};
  cuuint32_t estr[2] = {1, 1};
  const CUtensorMapSwizzle sw = span_bytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                : span_bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                                   : CU_TENSOR_MAP_SWIZZLE_32B;
  CUresult r = get_encode()(m, eb == 2 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, base,
                            dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
                            CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

void gemm_splitk_reduce(const TcEpilogue& ep, int M, int N, int out_bf16, cudaStream_t st) {
  const int64_t total = (int64_t)M * N;
  const unsigned grid = (unsigned)std::min<int64_t>((total + 255) / 256, 1184);
  if (out_bf16)
    launch_pdl(gemm_splitk_reduce_kernel<__nv_bfloat16>, dim3(grid), dim3(256), 0, st, (const float*)ep.ws, ep.bias,
               (__nv_bfloat16*)ep.out, M, N, ep.ldo, ep.splits, ep.act);
  else
    launch_pdl(gemm_splitk_reduce_kernel<float>, dim3(grid), dim3(256), 0, st, (const float*)ep.ws, ep.bias,
               (float*)ep.out, M, N, ep.ldo, ep.splits, ep.act);
}

int tc_splitk(int M, int N, int K, int bn, int num_sms) {
  static const bool off = getenv("DUET_SPLITK") && atoi(getenv("DUET_SPLITK")) == 0;
  const int tiles = ((M + BM - 1) / BM) * ((N + bn - 1) / bn);
  const int nk = (K + BK - 1) / BK;
  // only long K pays for the extra reduce launch (~3 us): measured on MT-DNN at batch 1, FFN2
  // (K = 3072, 48 k-blocks) 13.0 -> 8.4 us, but QKV / out / FFN1 (12 k-blocks) 4.9-5.5 -> 7.2-9.6 us
  if (off || tiles * 2 > num_sms || nk < 32) return 1;
  int splits = std::min(num_sms / tiles, nk / 2);
  if (splits < 2) return 1;
  const int per = (nk + splits - 1) / splits;
  return (nk + per - 1) / per;  // every split non-empty
}

int tc_pick_bn(int M, int N, int num_sms) {
  // Smallest-waste tile width that still fills the SMs: prefer the widest BN whose tile count
  // reaches the SM count; else the narrowest (most CTAs).
  const int cands[] = {256, 128, 64, 32};
  int mt = (M + BM - 1) / BM;
  for (int bn : cands) {
    if (bn > 128 && N < 256) continue;
    int tiles = mt * ((N + bn - 1) / bn);
    if (tiles >= num_sms) return bn;
  }
  return N <= 16 ? 16 : 32;
}

void gemm_tc(const void* A, const void* W, int M, int N, int K, int bn, const TcEpilogue& ep, int epi,
             int out_bf16, cudaStream_t st) {
  CUtensorMap ta = make_tmap_bf16_2d(A, M, K, BM);
  CUtensorMap tw = make_tmap_bf16_2d(W, N, K, bn);
  gemm_tc_maps(ta, tw, M, N, K, bn, ep, epi, out_bf16, st);
}

void gemm_tc_maps(const CUtensorMap& ta, const CUtensorMap& tw, int M, int N, int K, int bn, const TcEpilogue& ep,
                  int epi, int out_bf16, cudaStream_t st, const CUtensorMap* tx) {
  const CUtensorMap& tmx = tx ? *tx : ta;
#define DUET_TC_CASE(BNV)                                                        \
  case BNV:                                                                      \
    if (epi == EPI_BIAS_ACT) {                                                   \
      if (out_bf16)                                                              \
        launch_tc<BNV, EPI_BIAS_ACT, __nv_bfloat16>(ta, tw, tmx, ep, M, N, K, st);    \
      else                                                                       \
        launch_tc<BNV, EPI_BIAS_ACT, float>(ta, tw, tmx, ep, M, N, K, st);            \
      return;                                                                    \
    }                                                                            \
    break;
  switch (bn) {
    DUET_TC_CASE(16)
    DUET_TC_CASE(32)
    DUET_TC_CASE(64)
    DUET_TC_CASE(128)
    DUET_TC_CASE(256)
  }
#undef DUET_TC_CASE
  if (epi == EPI_LSTM) {
    if (bn == 128) return launch_tc<128, EPI_LSTM, __nv_bfloat16>(ta, tw, tmx, ep, M, N, K, st);
    if (bn == 256) return launch_tc<256, EPI_LSTM, __nv_bfloat16>(ta, tw, tmx, ep, M, N, K, st);
    if (bn == 64) return launch_tc<64, EPI_LSTM, __nv_bfloat16>(ta, tw, tmx, ep, M, N, K, st);
  }
  if (epi == EPI_GRU) {
    if (bn == 128) return launch_tc<128, EPI_GRU, __nv_bfloat16>(ta, tw, tmx, ep, M, N, K, st);
    if (bn == 256) return launch_tc<256, EPI_GRU, __nv_bfloat16>(ta, tw, tmx, ep, M, N, K, st);
    if (bn == 64) return launch_tc<64, EPI_GRU, __nv_bfloat16>(ta, tw, tmx, ep, M, N, K, st);
  }
  fail(DUET_EUNSUPPORTED, "no tcgen05 tile for bn=" + std::to_string(bn) + " epi=" + std::to_string(epi));
}

}  // namespace duet
