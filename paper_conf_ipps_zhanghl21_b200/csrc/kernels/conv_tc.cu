// Implicit-GEMM convolution on tcgen05 (R-27).
//
//   out[m, co] = act( sum_k A[m, k] * Wf[co, k] + bias[co] (+ res[m, co]) )
//   m = (n, ho, wo) output pixel (NHWC), k = (r, s, c) filter tap x input channel
//
// The A operand (im2col) is never materialised: 4 producer warps (thread t <-> tile row t) copy
// each k-block's 64 channels of the input pixel that row/tap needs straight into the
// SWIZZLE_128B K-major layout UMMA reads (16-B cp.async with zero-fill for the padding halo; a
// scalar gather path covers C % 64 != 0, i.e. the 3-channel stem), then fence the async proxy and
// arrive on the stage's mbarrier.  The BN-folded weights [Co, Kp] (K padded to 64 at build) stream
// in by TMA.  One thread issues UMMA 128 x BN x 16 into TMEM; 4 epilogue warps add the folded BN
// bias, the optional residual, apply ReLU and store bf16 NHWC.
#include "../common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace duet {

namespace {

constexpr int CBM = 128;
constexpr int CBK = 64;
constexpr int CA_BYTES = CBM * CBK * 2;
constexpr int LAG = 2;  // cp.async groups kept in flight per producer thread

template <int BN>
struct ConvCfg {
  static constexpr int B_BYTES = BN * CBK * 2;
  static constexpr int STAGE = CA_BYTES + B_BYTES;
  static constexpr int STAGES = (192 * 1024) / STAGE > 8 ? 8 : (192 * 1024) / STAGE;
  static constexpr int TMEM_COLS = BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : 256;
  static constexpr int SMEM = STAGES * STAGE + 1024 + 512 + BN * 4;
};

__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

struct ConvArgs {
  const __nv_bfloat16* x;
  const float* bias;
  const __nv_bfloat16* res;
  __nv_bfloat16* y;
  ConvShape s;
  int K;   // kh * kw * C (true reduction length)
  int act;
};

template <int BN, bool VEC>
__global__ void __launch_bounds__(320, 1) conv_tc_kernel(const __grid_constant__ CUtensorMap tmW, const ConvArgs a) {
  using C = ConvCfg<BN>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::STAGES * CA_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(sB + C::STAGES * C::B_BYTES);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tmem_full = empty + C::STAGES;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_full + 1);
  float* s_bias = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(full) + 512);

  const ConvShape& s = a.s;
  const int warp = ptx::warp_id();
  const int lane = threadIdx.x & 31;
  const int64_t M = (int64_t)s.N * s.Ho * s.Wo;
  const int n0 = blockIdx.x * BN;
  const int64_t m0 = (int64_t)blockIdx.y * CBM;
  const int nk = (a.K + CBK - 1) / CBK;

  if (threadIdx.x == 128) {
    ptx::tma_prefetch(&tmW);
    for (int i = 0; i < C::STAGES; ++i) {
      ptx::mbar_init(&full[i], 128 + 1);
      ptx::mbar_init(&empty[i], 1);
    }
    ptx::mbar_init(tmem_full, 1);
    ptx::fence_mbar_init();
  }
  if (warp == 5) {
    ptx::tmem_alloc(tmem_slot, C::TMEM_COLS);
    ptx::tmem_relinquish();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp < 4) {
    // ---------------- im2col producers: thread t owns tile row t ----------------
    const int t = threadIdx.x;
    const int64_t m = m0 + t;
    const bool mvalid = m < M;
    int nn = 0, ho = 0, wo = 0;
    if (mvalid) {
      wo = (int)(m % s.Wo);
      int64_t q = m / s.Wo;
      ho = (int)(q % s.Ho);
      nn = (int)(q / s.Ho);
    }
    const int hbase = ho * s.stride - s.pad, wbase = wo * s.stride - s.pad;
    const int sw = t & 7;
    for (int kb = 0; kb < nk; ++kb) {
      const int st = kb % C::STAGES;
      if (kb >= C::STAGES) ptx::mbar_wait(&empty[st], ((kb / C::STAGES) - 1) & 1);
      const uint32_t row_smem = ptx::smem_u32(sA + st * CA_BYTES + t * 128);
      if constexpr (VEC) {
        const int cb = s.C / 64;
        const int tap = kb / cb, c0 = (kb - tap * cb) * 64;
        const int r = tap / s.kw, q = tap - r * s.kw;
        const int hi = hbase + r, wi = wbase + q;
        const bool ok = mvalid && hi >= 0 && hi < s.H && wi >= 0 && wi < s.W;
        const __nv_bfloat16* src = a.x + ((((int64_t)nn * s.H + (ok ? hi : 0)) * s.W + (ok ? wi : 0)) * s.C + c0);
#pragma unroll
        for (int j = 0; j < 8; ++j) cp_async16(row_smem + ((j ^ sw) << 4), src + j * 8, ok ? 16u : 0u);
        cp_async_commit();
        if (kb >= LAG) {
          cp_async_wait<LAG>();
          fence_proxy_async();
          ptx::mbar_arrive(&full[(kb - LAG) % C::STAGES]);
        }
      } else {
        // generic gather (C % 64 != 0): 64 scalar taps of this row, packed to 8 x 16 B
        uint32_t w[32];
#pragma unroll
        for (int e2 = 0; e2 < 32; ++e2) {
          uint16_t h2[2];
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int k = kb * CBK + 2 * e2 + h;
            uint16_t v = 0;
            if (mvalid && k < a.K) {
              const int c = k % s.C, tap = k / s.C;
              const int r = tap / s.kw, q = tap - r * s.kw;
              const int hi = hbase + r, wi = wbase + q;
              if (hi >= 0 && hi < s.H && wi >= 0 && wi < s.W)
                v = reinterpret_cast<const uint16_t*>(a.x)[(((int64_t)nn * s.H + hi) * s.W + wi) * s.C + c];
            }
            h2[h] = v;
          }
          w[e2] = (uint32_t)h2[0] | ((uint32_t)h2[1] << 16);
        }
#pragma unroll
        for (int j = 0; j < 8; ++j)
          asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(row_smem + ((j ^ sw) << 4)), "r"(w[4 * j]),
                       "r"(w[4 * j + 1]), "r"(w[4 * j + 2]), "r"(w[4 * j + 3])
                       : "memory");
        fence_proxy_async();
        ptx::mbar_arrive(&full[st]);
      }
    }
    if constexpr (VEC) {
      cp_async_wait<0>();
      fence_proxy_async();
      for (int kb = (nk > LAG ? nk - LAG : 0); kb < nk; ++kb) ptx::mbar_arrive(&full[kb % C::STAGES]);
    }
  } else if (warp == 4) {
    if (lane == 0) {
      for (int kb = 0; kb < nk; ++kb) {
        const int st = kb % C::STAGES;
        if (kb >= C::STAGES) ptx::mbar_wait(&empty[st], ((kb / C::STAGES) - 1) & 1);
        ptx::mbar_arrive_expect_tx(&full[st], C::B_BYTES);
        ptx::tma_load_2d(&tmW, &full[st], sB + st * C::B_BYTES, kb * CBK, n0);
      }
    }
  } else if (warp == 5) {
    if (lane == 0) {
      constexpr uint32_t idesc = ptx::idesc_bf16(CBM, BN);
      for (int kb = 0; kb < nk; ++kb) {
        const int st = kb % C::STAGES;
        ptx::mbar_wait(&full[st], (kb / C::STAGES) & 1);
        ptx::tc_fence_after();
        const uint32_t a_base = ptx::smem_u32(sA + st * CA_BYTES);
        const uint32_t b_base = ptx::smem_u32(sB + st * C::B_BYTES);
#pragma unroll
        for (int k = 0; k < CBK / 16; ++k)
          ptx::umma_bf16(tmem, ptx::desc_sw128(a_base + k * 32), ptx::desc_sw128(b_base + k * 32), idesc,
                         (kb | k) != 0);
        ptx::umma_commit(&empty[st]);
      }
      ptx::umma_commit(tmem_full);
    }
  } else {
    // ---------------- epilogue warps 6..9 ----------------
    const int et = threadIdx.x - 192;
    for (int c = et; c < BN; c += 128) s_bias[c] = (n0 + c < s.Co) ? a.bias[n0 + c] : 0.0f;
    asm volatile("bar.sync 1, 128;" ::: "memory");
    const int qd = warp & 3;
    const int64_t row = m0 + qd * 32 + lane;
    ptx::mbar_wait(tmem_full, 0);
    ptx::tc_fence_after();
    const uint32_t tq = tmem + ((uint32_t)(qd * 32) << 16);
    __nv_bfloat16* out = a.y + row * s.Co;
    const __nv_bfloat16* res = a.res ? a.res + row * s.Co : nullptr;
#pragma unroll 1
    for (int c = 0; c < BN / 16; ++c) {
      float v[16];
      ptx::tmem_ld16(tq + c * 16, v);
      const int col0 = n0 + c * 16;
      if (row < M && col0 < s.Co) {
        if (res && col0 + 16 <= s.Co) {
          uint4 r0 = *reinterpret_cast<const uint4*>(res + col0);
          uint4 r1 = *reinterpret_cast<const uint4*>(res + col0 + 8);
          const __nv_bfloat16* rb0 = reinterpret_cast<const __nv_bfloat16*>(&r0);
          const __nv_bfloat16* rb1 = reinterpret_cast<const __nv_bfloat16*>(&r1);
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            v[i] += __bfloat162float(rb0[i]);
            v[8 + i] += __bfloat162float(rb1[i]);
          }
        } else if (res) {
#pragma unroll
          for (int i = 0; i < 16; ++i)
            if (col0 + i < s.Co) v[i] += __bfloat162float(res[col0 + i]);
        }
#pragma unroll
        for (int i = 0; i < 16; ++i) v[i] = apply_act(v[i] + s_bias[c * 16 + i], a.act);
        store_row16_any(out + col0, v, s.Co - col0);
      }
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 5) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, C::TMEM_COLS);
  }
}

template <int BN, bool VEC>
void launch_conv(const CUtensorMap& tw, const ConvArgs& a, cudaStream_t st) {
  using C = ConvCfg<BN>;
  auto kern = conv_tc_kernel<BN, VEC>;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM));
    attr = true;
  }
  const int64_t M = (int64_t)a.s.N * a.s.Ho * a.s.Wo;
  dim3 grid((a.s.Co + BN - 1) / BN, (unsigned)((M + CBM - 1) / CBM));
  kern<<<grid, 320, C::SMEM, st>>>(tw, a);
  CK(cudaGetLastError());
}

}  // namespace

int conv_tc_pick_bn(const ConvShape& s, int sms) {
  const int64_t mt = ((int64_t)s.N * s.Ho * s.Wo + CBM - 1) / CBM;
  for (int bn : {256, 128, 64}) {
    if (bn > s.Co && bn > 64) continue;
    if (mt * ((s.Co + bn - 1) / bn) * 5 >= (int64_t)sms * 4) return bn;
  }
  return 64;
}

void conv_tc(const CUtensorMap& tw, const void* x, const float* bias, const void* residual, void* y,
             const ConvShape& s, int K, int act, int bn, cudaStream_t st) {
  ConvArgs a{(const __nv_bfloat16*)x, bias, (const __nv_bfloat16*)residual, (__nv_bfloat16*)y, s, K, act};
  const bool vec = s.C % 64 == 0 && ((uintptr_t)x % 16) == 0;
  switch (bn) {
    case 64: return vec ? launch_conv<64, true>(tw, a, st) : launch_conv<64, false>(tw, a, st);
    case 128: return vec ? launch_conv<128, true>(tw, a, st) : launch_conv<128, false>(tw, a, st);
    case 256: return vec ? launch_conv<256, true>(tw, a, st) : launch_conv<256, false>(tw, a, st);
  }
  fail(DUET_EUNSUPPORTED, "conv_tc: bn must be 64, 128 or 256");
}

}  // namespace duet
