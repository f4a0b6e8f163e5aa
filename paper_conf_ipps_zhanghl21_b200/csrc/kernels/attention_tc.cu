// MT-DNN self-attention on tcgen05 (Fig. 3: the shared
// Transformer encoder; QK^T and PV are contractions and belong on the tensor
// cores).  bf16, head dim 64, sequences of at most 128 tokens (BERT-base / MT-DNN at S = 128).
//
// One CTA per (sequence, head), 4 warps, one query row per thread (= TMEM lane):
//   TMA      Q, K, V tiles [128 rows x 64] of the head from qkv [B*S, 3H] (SWIZZLE_128B; rows past
//            the tensor zero-filled, rows of the next sequence masked below)
//   UMMA 1   S = Q K^T      A = Q (K-major), B = K (K-major)         128 x 128 x 64 -> TMEM cols [0,128)
//   softmax  each thread reads its 128 scores from TMEM, scale 1/sqrt(dh), keys >= S masked,
//            p = exp2((s - max) log2 e) in fp32, P (bf16, unnormalised) written to SMEM in the
//            SWIZZLE_128B K-major layout of an A operand; the row sum stays in a register
//   UMMA 2   O = P V        A = P (K-major, K = 128 keys), B = V as loaded (row = key, 64 dh
//            values contiguous): the MN-major B layout (instruction descriptor "transpose B")
//                                                                  128 x 64 x 128 -> TMEM cols [128,192)
//   epilogue O / rowsum -> bf16, the valid query rows stored to out [B*S, H]
#include <cudaTypedefs.h>

#include "../common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace duet {

namespace {

constexpr int AT_ROWS = 128;
constexpr int AT_TILE = AT_ROWS * 128;  // one [128 x 64] bf16 tile, 16 KB

__global__ void __launch_bounds__(128, 1)
    attention_tc_kernel(const __grid_constant__ CUtensorMap tq, __nv_bfloat16* __restrict__ out, int S, int heads) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sK = sQ + AT_TILE;
  uint8_t* sV = sK + AT_TILE;
  uint8_t* sP = sV + AT_TILE;  // 2 x [128 x 64] (keys 0-63, 64-127)
  uint64_t* bars = reinterpret_cast<uint64_t*>(sP + 2 * AT_TILE);
  uint64_t* tma_bar = bars;
  uint64_t* s_bar = bars + 1;
  uint64_t* o_bar = bars + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 3);

  const int warp = ptx::warp_id();
  const int lane = threadIdx.x & 31;
  const int b = blockIdx.x / heads, h = blockIdx.x % heads;
  const int H = heads * 64;
  const int m = threadIdx.x;  // query row within the sequence = TMEM lane

  if (threadIdx.x == 0) {
    ptx::tma_prefetch(&tq);
    ptx::mbar_init(tma_bar, 1);
    ptx::mbar_init(s_bar, 1);
    ptx::mbar_init(o_bar, 1);
    ptx::fence_mbar_init();
  }
  ptx::pdl_wait();
  if (warp == 0) {
    ptx::tmem_alloc(tmem_slot, 256);  // S: 128 columns, O: 64 columns
    ptx::tmem_relinquish();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  ptx::pdl_trigger();

  if (threadIdx.x == 0) {
    ptx::mbar_arrive_expect_tx(tma_bar, 3 * AT_TILE);
    const int row = b * S;
    ptx::tma_load_2d(&tq, tma_bar, sQ, h * 64, row);
    ptx::tma_load_2d(&tq, tma_bar, sK, H + h * 64, row);
    ptx::tma_load_2d(&tq, tma_bar, sV, 2 * H + h * 64, row);
  }
  if (warp == 0) {
    ptx::mbar_wait(tma_bar, 0);
    ptx::tc_fence_after();
    constexpr uint32_t idesc = ptx::idesc_bf16(AT_ROWS, AT_ROWS);
    const uint64_t dq = ptx::desc_sw128(ptx::smem_u32(sQ));
    const uint64_t dk = ptx::desc_sw128(ptx::smem_u32(sK));
#pragma unroll
    for (int k = 0; k < 4; ++k) ptx::umma_bf16_elect(tmem, dq + 2 * k, dk + 2 * k, idesc, k != 0);
    ptx::umma_commit_elect(s_bar);
  }

  // ---- softmax over the keys of row m ----
  ptx::mbar_wait(s_bar, 0);
  ptx::tc_fence_after();
  const uint32_t trow = tmem + ((uint32_t)(warp * 32) << 16);
  float s[128];
#pragma unroll
  for (int c = 0; c < 8; ++c) ptx::tmem_ld16(trow + 16 * c, s + 16 * c);
  const float kscale = 0.125f * 1.4426950408889634f;  // 1/sqrt(64) * log2(e)
  float mx = -INFINITY;
#pragma unroll
  for (int j = 0; j < 128; ++j) {
    s[j] = j < S ? s[j] * kscale : -INFINITY;
    mx = fmaxf(mx, s[j]);
  }
  // the row sum is taken over the bf16-rounded probabilities the second UMMA multiplies, so the
  // normalisation matches the numerator (no systematic bias from rounding P)
  float sum = 0.0f;
#pragma unroll
  for (int j = 0; j < 128; ++j) {
    s[j] = __bfloat162float(__float2bfloat16_rn(exp2f(s[j] - mx)));
    sum += s[j];
  }
  // P row m, keys j: atom a = j / 64, 16-byte chunk c = (j % 64) / 8 at position c ^ (m % 8)
#pragma unroll
  for (int a = 0; a < 2; ++a)
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      uint32_t w[4];
#pragma unroll
      for (int p = 0; p < 4; ++p) {
        __nv_bfloat162 v = __floats2bfloat162_rn(s[a * 64 + c * 8 + 2 * p], s[a * 64 + c * 8 + 2 * p + 1]);
        w[p] = *reinterpret_cast<uint32_t*>(&v);
      }
      uint8_t* dst = sP + a * AT_TILE + (m >> 3) * 1024 + (m & 7) * 128 + ((c ^ (m & 7)) << 4);
      *reinterpret_cast<uint4*>(dst) = make_uint4(w[0], w[1], w[2], w[3]);
    }
  ptx::fence_async_smem();  // generic-proxy P stores -> visible to the tensor core (async proxy)
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    ptx::tc_fence_after();
    // O = P V: B = V in the MN-major layout (rows = keys, 64 dh values contiguous): an 8-key group
    // is 1024 B, a 16-key UMMA step advances 2048 B; transpose-B bit 16 of the instruction descriptor
    constexpr uint32_t idesc = ptx::idesc_bf16(AT_ROWS, 64) | (1u << 16);
    const uint64_t dp = ptx::desc_sw128(ptx::smem_u32(sP));
    const uint64_t dv = ptx::desc_sw128(ptx::smem_u32(sV));
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const uint64_t da = dp + (uint64_t)(((k >> 2) * AT_TILE) >> 4) + 2 * (k & 3);
      const uint64_t db = dv + (uint64_t)((k * 2048) >> 4);
      ptx::umma_bf16_elect(tmem + 128, da, db, idesc, k != 0);
    }
    ptx::umma_commit_elect(o_bar);
  }
  ptx::mbar_wait(o_bar, 0);
  ptx::tc_fence_after();
  float o[64];
  ptx::tmem_ld64(trow + 128, o);
  if (m < S) {
    const float inv = 1.0f / sum;
    __nv_bfloat16* dst = out + ((int64_t)b * S + m) * H + h * 64;
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      uint32_t w[4];
#pragma unroll
      for (int p = 0; p < 4; ++p) {
        __nv_bfloat162 v = __floats2bfloat162_rn(o[c * 8 + 2 * p] * inv, o[c * 8 + 2 * p + 1] * inv);
        w[p] = *reinterpret_cast<uint32_t*>(&v);
      }
      *reinterpret_cast<uint4*>(dst + c * 8) = make_uint4(w[0], w[1], w[2], w[3]);
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, 256);
  }
}

}  // namespace

bool attention_tc_ok(int S, int dh, int bf16) { return bf16 && dh == 64 && S >= 1 && S <= 128; }

void attention_tc(const void* qkv, void* out, int B, int S, int heads, cudaStream_t st) {
  const int H = heads * 64;
  if (((uintptr_t)qkv & 15) || ((uintptr_t)out & 15)) fail(DUET_EUNSUPPORTED, "attention_tc: 16-B aligned tensors");
  CUtensorMap tq = make_tmap_bf16_2d(qkv, (int64_t)B * S, 3 * H, AT_ROWS);
  constexpr int smem = 1024 + 5 * AT_TILE + 64;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(attention_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    attr = true;
  }
  launch_pdl_if(pdl_on(true), attention_tc_kernel, dim3(B * heads), dim3(128), smem, st, tq, (__nv_bfloat16*)out, S,
                heads);
}

}  // namespace duet
