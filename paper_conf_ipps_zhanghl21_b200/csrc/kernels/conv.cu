// Convolution as implicit GEMM: M = N*Ho*Wo output pixels,
// N = Co, K = kh*kw*C in (r, s, c) order = the NHWC weight layout [Co, kh, kw, C].  BN is folded
// into the weights and a per-channel bias once at program build (fold_bn); the epilogue adds
// bias, an optional residual, and the activation.
//
// This file holds the CUDA-core implicit GEMM (fp32 parity path and the generic fallback).
#include <cuda_bf16.h>

#include "kernels.h"
#include "ptx.cuh"

namespace duet {

namespace {

__device__ __forceinline__ float ldx(const void* p, int64_t i, int bf16) {
  return bf16 ? __bfloat162float(reinterpret_cast<const __nv_bfloat16*>(p)[i]) : reinterpret_cast<const float*>(p)[i];
}
__device__ __forceinline__ void stx(void* p, int64_t i, float v, int bf16) {
  if (bf16)
    reinterpret_cast<__nv_bfloat16*>(p)[i] = __float2bfloat16_rn(v);
  else
    reinterpret_cast<float*>(p)[i] = v;
}

__global__ void __launch_bounds__(256) conv_simt_kernel(const void* __restrict__ x, const void* __restrict__ Wf,
                                                        const float* __restrict__ bias, const void* __restrict__ res,
                                                        void* __restrict__ y, int bf16, ConvShape s, int act) {
  __shared__ float As[16][64 + 4];
  __shared__ float Ws[16][64 + 4];
  const int64_t M = (int64_t)s.N * s.Ho * s.Wo;
  const int Nn = s.Co;
  const int K = s.kh * s.kw * s.C;
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  const int64_t m0 = (int64_t)blockIdx.y * 64;
  const int n0 = blockIdx.x * 64;
  float acc[4][4] = {};
  for (int k0 = 0; k0 < K; k0 += 16) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      int e = threadIdx.x + i * 256;
      int r = e >> 4, kk = e & 15;
      int gk = k0 + kk;
      int64_t gm = m0 + r;
      float av = 0.0f;
      if (gm < M && gk < K) {
        int c = gk % s.C;
        int t = gk / s.C;
        int q = t % s.kw, p = t / s.kw;
        int wo = (int)(gm % s.Wo);
        int64_t t2 = gm / s.Wo;
        int ho = (int)(t2 % s.Ho);
        int n = (int)(t2 / s.Ho);
        int hi = ho * s.stride - s.pad + p, wi = wo * s.stride - s.pad + q;
        if (hi >= 0 && hi < s.H && wi >= 0 && wi < s.W) av = ldx(x, (((int64_t)n * s.H + hi) * s.W + wi) * s.C + c, bf16);
      }
      As[kk][r] = av;
      int gn = n0 + r;
      Ws[kk][r] = (gn < Nn && gk < K) ? ldx(Wf, (int64_t)gn * K + gk, bf16) : 0.0f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < 16; ++kk) {
      float a[4], w[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        a[i] = As[kk][ty * 4 + i];
        w[i] = Ws[kk][tx * 4 + i];
      }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], w[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    int64_t m = m0 + ty * 4 + i;
    if (m >= M) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      int n = n0 + tx * 4 + j;
      if (n >= Nn) continue;
      float v = acc[i][j] + bias[n];
      if (res) v += ldx(res, m * Nn + n, bf16);
      stx(y, m * Nn + n, apply_act(v, act), bf16);
    }
  }
}

__global__ void fold_bn_kernel(const void* W, int bf16, const float* g, const float* beta, const float* mean,
                               const float* var, void* Wf, float* bias, int Co, int64_t per_co, int64_t ldw) {
  int64_t total = (int64_t)Co * ldw;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    int co = (int)(i / ldw);
    int64_t k = i - (int64_t)co * ldw;
    float sc = g[co] / sqrtf(var[co] + 1e-5f);
    stx(Wf, i, k < per_co ? ldx(W, (int64_t)co * per_co + k, bf16) * sc : 0.0f, bf16);
    if (k == 0) bias[co] = beta[co] - mean[co] * sc;
  }
}

// one thread per output row m: decode (n, ho, wo) once, walk k = (r, q, c) with incremental
// counters (no per-element division), write the row as 16-B stores
__global__ void im2col_kernel(const __nv_bfloat16* __restrict__ x, __nv_bfloat16* __restrict__ cols, ConvShape s,
                              int ldk) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  const int K = s.kh * s.kw * s.C;
  const int M = s.N * s.Ho * s.Wo;
  const uint16_t* xs = reinterpret_cast<const uint16_t*>(x);
  for (int m = blockIdx.x * blockDim.x + threadIdx.x; m < M; m += gridDim.x * blockDim.x) {
    const int wo = m % s.Wo;
    const int q0 = m / s.Wo;
    const int ho = q0 % s.Ho;
    const int n = q0 / s.Ho;
    const int hb = ho * s.stride - s.pad, wb = wo * s.stride - s.pad;
    uint4* dst = reinterpret_cast<uint4*>(cols + (int64_t)m * ldk);
    int c = 0, q = 0, r = 0;
    for (int k0 = 0; k0 < ldk; k0 += 8) {
      uint32_t w[4];
#pragma unroll
      for (int e = 0; e < 8; e += 2) {
        uint32_t pair = 0;
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int k = k0 + e + h;
          uint32_t v = 0;
          if (k < K) {
            const int hi = hb + r, wi = wb + q;
            if ((unsigned)hi < (unsigned)s.H && (unsigned)wi < (unsigned)s.W)
              v = xs[(((int64_t)n * s.H + hi) * s.W + wi) * s.C + c];
            if (++c == s.C) {
              c = 0;
              if (++q == s.kw) {
                q = 0;
                ++r;
              }
            }
          }
          pair |= v << (16 * h);
        }
        w[e / 2] = pair;
      }
      dst[k0 / 8] = make_uint4(w[0], w[1], w[2], w[3]);
    }
  }
}

}  // namespace

void im2col(const void* x, void* cols, const ConvShape& s, int64_t ldk, cudaStream_t st) {
  const int64_t M = (int64_t)s.N * s.Ho * s.Wo;
  if (!M) return;
  if (M >= INT32_MAX || ldk % 8) fail(DUET_EUNSUPPORTED, "im2col: M < 2^31 and ldk % 8 == 0 required");
  launch_plain(im2col_kernel, dim3(grid_for(M, 128, 16)), dim3(128), 0, st, (const __nv_bfloat16*)x, (__nv_bfloat16*)cols, s,
             (int)ldk);
  CK(cudaGetLastError());
}

void conv_fwd(const void* x, const void* Wf, const float* bias, const void* residual, void* y, int bf16,
              const ConvShape& s, int act, cudaStream_t st) {
  int64_t M = (int64_t)s.N * s.Ho * s.Wo;
  if (M == 0) return;
  dim3 grid((s.Co + 63) / 64, (unsigned)((M + 63) / 64));
  conv_simt_kernel<<<grid, 256, 0, st>>>(x, Wf, bias, residual, y, bf16, s, act);
  CK(cudaGetLastError());
}

void fold_bn(const void* W, int bf16, const float* g, const float* beta, const float* mean, const float* var, void* Wf,
             float* bias, int Co, int64_t per_co, int64_t ldw, cudaStream_t st) {
  fold_bn_kernel<<<grid_for((int64_t)Co * ldw, 256), 256, 0, st>>>(W, bf16, g, beta, mean, var, Wf, bias, Co,
                                                                  per_co, ldw);
  CK(cudaGetLastError());
}

}  // namespace duet
