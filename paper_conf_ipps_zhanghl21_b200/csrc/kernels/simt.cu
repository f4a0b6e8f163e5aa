// CUDA-core kernels: the fp32 parity path of the dense contractions (tcgen05 has no fp32 kind;
// SURVEY.md §7 "fp32 parity at 1e-5"), the fused small-M MLP (c1 at batch 1 is launch-bound:
// one CTA runs every layer), and the fp32 RNN step.
#include <cuda_bf16.h>

#include "kernels.h"
#include "ptx.cuh"

namespace duet {

namespace {

template <typename T>
__device__ __forceinline__ float ldf(const void* p, int64_t i) {
  return to_f(reinterpret_cast<const T*>(p)[i]);
}
__device__ __forceinline__ float ldx(const void* p, int64_t i, int bf16) {
  return bf16 ? __bfloat162float(reinterpret_cast<const __nv_bfloat16*>(p)[i]) : reinterpret_cast<const float*>(p)[i];
}
__device__ __forceinline__ void stx(void* p, int64_t i, float v, int bf16) {
  if (bf16)
    reinterpret_cast<__nv_bfloat16*>(p)[i] = __float2bfloat16_rn(v);
  else
    reinterpret_cast<float*>(p)[i] = v;
}

// 64 x 64 output tile, BK = 16, 256 threads, 4 x 4 outputs per thread.
template <typename TX, typename TW>
__global__ void __launch_bounds__(256) gemm_simt_kernel(const TX* __restrict__ X, const TW* __restrict__ W,
                                                        const float* __restrict__ bias, void* __restrict__ Y,
                                                        int y_bf16, int M, int N, int K, int act) {
  __shared__ float As[16][64 + 4];
  __shared__ float Ws[16][64 + 4];
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  const int m0 = blockIdx.y * 64, n0 = blockIdx.x * 64;
  float acc[4][4] = {};
  for (int k0 = 0; k0 < K; k0 += 16) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      int e = threadIdx.x + i * 256;  // 0..1023
      int r = e >> 4, k = e & 15;
      int gm = m0 + r, gk = k0 + k, gn = n0 + r;
      As[k][r] = (gm < M && gk < K) ? to_f(X[(int64_t)gm * K + gk]) : 0.0f;
      Ws[k][r] = (gn < N && gk < K) ? to_f(W[(int64_t)gn * K + gk]) : 0.0f;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < 16; ++k) {
      float a[4], w[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        a[i] = As[k][ty * 4 + i];
        w[i] = Ws[k][tx * 4 + i];
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
    int m = m0 + ty * 4 + i;
    if (m >= M) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      int n = n0 + tx * 4 + j;
      if (n >= N) continue;
      float v = acc[i][j] + (bias ? bias[n] : 0.0f);
      stx(Y, (int64_t)m * N + n, apply_act(v, act), y_bf16);
    }
  }
}

struct MlpArgs {
  const void* W[8];
  const float* b[8];
  int dims[9];
  int L;
};

// One CTA per block of up to 4 rows; activations ping-pong in shared memory (fp32).  32 warps;
// each warp computes 2 outputs at a time with independent loads in flight (latency-bound at M = 1).
__global__ void __launch_bounds__(1024) mlp_small_kernel(const void* __restrict__ X, int bf16, MlpArgs a,
                                                         void* __restrict__ Y, int y_bf16, int M, int act, int last_act,
                                                         int maxd) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  extern __shared__ float sm[];
  const int R = 4;
  float* buf0 = sm;
  float* buf1 = sm + R * maxd;
  const int r0 = blockIdx.x * R;
  const int nr = min(R, M - r0);
  for (int i = threadIdx.x; i < nr * a.dims[0]; i += blockDim.x) {
    int r = i / a.dims[0], k = i - r * a.dims[0];
    buf0[r * maxd + k] = ldx(X, (int64_t)(r0 + r) * a.dims[0] + k, bf16);
  }
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  float* in = buf0;
  float* out = buf1;
  for (int l = 0; l < a.L; ++l) {
    const int K = a.dims[l], N = a.dims[l + 1];
    const bool last = (l + 1 == a.L);
    const int total = nr * N;
    for (int o = warp * 2; o < total; o += nw * 2) {
      const int o1 = o + 1 < total ? o + 1 : o;
      const int ra = o / N, na = o - ra * N, rb = o1 / N, nb = o1 - rb * N;
      float sa = 0.0f, sb = 0.0f;
      for (int k = lane; k < K; k += 32) {
        const float wa = ldx(a.W[l], (int64_t)na * K + k, bf16);
        const float wb = ldx(a.W[l], (int64_t)nb * K + k, bf16);
        sa = fmaf(in[ra * maxd + k], wa, sa);
        sb = fmaf(in[rb * maxd + k], wb, sb);
      }
      sa = warp_sum(sa);
      sb = warp_sum(sb);
      if (lane == 0) {
        const float va = apply_act(sa + a.b[l][na], last ? last_act : act);
        const float vb = apply_act(sb + a.b[l][nb], last ? last_act : act);
        if (last) {
          stx(Y, (int64_t)(r0 + ra) * N + na, va, y_bf16);
          if (o1 != o) stx(Y, (int64_t)(r0 + rb) * N + nb, vb, y_bf16);
        } else {
          out[ra * maxd + na] = bf16 ? __bfloat162float(__float2bfloat16_rn(va)) : va;  // stored-dtype rounding
          if (o1 != o) out[rb * maxd + nb] = bf16 ? __bfloat162float(__float2bfloat16_rn(vb)) : vb;
        }
      }
    }
    __syncthreads();
    float* t = in;
    in = out;
    out = t;
  }
}

// fp32 RNN step (original PyTorch layout). Block: 32 units x 8 rows; K tiled by 32.
template <int G>
__global__ void __launch_bounds__(256) rnn_step_simt_kernel(const float* __restrict__ gx, const void* __restrict__ Whh,
                                                            int w_bf16, const float* __restrict__ bhn,
                                                            const void* __restrict__ h_prev, void* __restrict__ h_next,
                                                            int h_bf16, float* __restrict__ c_state, int M, int H) {
  __shared__ float hs[8][33];
  __shared__ float ws[G][32][33];
  const int tu = threadIdx.x & 31, tr = threadIdx.x >> 5;
  const int j = blockIdx.x * 32 + tu;
  const int b = blockIdx.y * 8 + tr;
  float acc[G] = {};
  for (int k0 = 0; k0 < H; k0 += 32) {
    {
      int kk = threadIdx.x & 31, rr = threadIdx.x >> 5;
      int gb = blockIdx.y * 8 + rr, gk = k0 + kk;
      hs[rr][kk] = (gb < M && gk < H) ? ldx(h_prev, (int64_t)gb * H + gk, h_bf16) : 0.0f;
    }
    for (int e = threadIdx.x; e < G * 32 * 32; e += 256) {
      int g = e / 1024, rem = e - g * 1024, u = rem >> 5, kk = rem & 31;
      int gj = blockIdx.x * 32 + u, gk = k0 + kk;
      ws[g][u][kk] = (gj < H && gk < H) ? ldx(Whh, (int64_t)(g * H + gj) * H + gk, w_bf16) : 0.0f;
    }
    __syncthreads();
#pragma unroll 8
    for (int kk = 0; kk < 32; ++kk) {
      float hv = hs[tr][kk];
#pragma unroll
      for (int g = 0; g < G; ++g) acc[g] = fmaf(hv, ws[g][tu][kk], acc[g]);
    }
    __syncthreads();
  }
  if (b >= M || j >= H) return;
  const float* gr = gx + (int64_t)b * G * H;
  float h;
  if (G == 4) {
    float ig = sigmoidf_acc(gr[j] + acc[0]);
    float fg = sigmoidf_acc(gr[H + j] + acc[1]);
    float gg = tanhf(gr[2 * H + j] + acc[2]);
    float og = sigmoidf_acc(gr[3 * H + j] + acc[3]);
    float c = fg * c_state[(int64_t)b * H + j] + ig * gg;
    c_state[(int64_t)b * H + j] = c;
    h = og * tanhf(c);
  } else {
    float r = sigmoidf_acc(gr[j] + acc[0]);
    float z = sigmoidf_acc(gr[H + j] + acc[1]);
    float n = tanhf(gr[2 * H + j] + r * (acc[2] + bhn[j]));
    h = (1.0f - z) * n + z * ldx(h_prev, (int64_t)b * H + j, h_bf16);
  }
  stx(h_next, (int64_t)b * H + j, h, h_bf16);
}

}  // namespace

// Narrow linear (N <= 8 outputs, the per-branch logit heads): one warp per row, the row streamed
// once with 16-byte loads (HBM-bound: M*K*esize bytes), W rows from L1, warp-shuffle reduction.
template <typename TX, typename TW>
__global__ void __launch_bounds__(256) linear_narrow_kernel(const TX* __restrict__ X, const TW* __restrict__ W,
                                                            const float* __restrict__ bias, void* __restrict__ Y,
                                                            int y_bf16, int M, int N, int K, int act) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  const int warps = blockDim.x >> 5, lane = threadIdx.x & 31;
  constexpr int V = 16 / sizeof(TX);  // elements per 16-byte vector of X
  const bool vec = (K % V == 0) && ((uintptr_t)X % 16 == 0);
  for (int m = blockIdx.x * warps + (threadIdx.x >> 5); m < M; m += gridDim.x * warps) {
    float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    const TX* xr = X + (int64_t)m * K;
    if (vec) {
      for (int k0 = lane * V; k0 < K; k0 += 32 * V) {
        const uint4 raw = __ldcs(reinterpret_cast<const uint4*>(xr + k0));
        const TX* xv = reinterpret_cast<const TX*>(&raw);
#pragma unroll
        for (int n = 0; n < 8; ++n) {
          if (n >= N) break;
          const TW* wr = W + (int64_t)n * K + k0;
#pragma unroll
          for (int i = 0; i < V; ++i) acc[n] = fmaf(to_f(xv[i]), to_f(__ldg(wr + i)), acc[n]);
        }
      }
    } else {
      for (int k = lane; k < K; k += 32) {
        const float xv = to_f(xr[k]);
#pragma unroll
        for (int n = 0; n < 8; ++n)
          if (n < N) acc[n] = fmaf(xv, to_f(W[(int64_t)n * K + k]), acc[n]);
      }
    }
#pragma unroll
    for (int n = 0; n < 8; ++n) {
      if (n >= N) break;
      const float v = warp_sum(acc[n]);
      if (lane == 0) {
        const float o = apply_act(v + (bias ? bias[n] : 0.0f), act);
        if (y_bf16) reinterpret_cast<__nv_bfloat16*>(Y)[(int64_t)m * N + n] = __float2bfloat16_rn(o);
        else reinterpret_cast<float*>(Y)[(int64_t)m * N + n] = o;
      }
    }
  }
}

void gemm_simt(const void* X, int x_bf16, const void* W, int w_bf16, const float* b, void* Y, int y_bf16, int M, int N,
               int K, int act, cudaStream_t st) {
  if (M == 0 || N == 0) return;
  if (N <= 8) {
    const dim3 g(grid_for((int64_t)M * 32, 256, 4));
    if (x_bf16 && w_bf16)
      launch_pdl(linear_narrow_kernel<__nv_bfloat16, __nv_bfloat16>, g, dim3(256), 0, st, (const __nv_bfloat16*)X,
                 (const __nv_bfloat16*)W, b, Y, y_bf16, M, N, K, act);
    else if (!x_bf16 && !w_bf16)
      launch_pdl(linear_narrow_kernel<float, float>, g, dim3(256), 0, st, (const float*)X, (const float*)W, b, Y, y_bf16,
                 M, N, K, act);
    else if (x_bf16)
      launch_pdl(linear_narrow_kernel<__nv_bfloat16, float>, g, dim3(256), 0, st, (const __nv_bfloat16*)X,
                 (const float*)W, b, Y, y_bf16, M, N, K, act);
    else
      launch_pdl(linear_narrow_kernel<float, __nv_bfloat16>, g, dim3(256), 0, st, (const float*)X,
                 (const __nv_bfloat16*)W, b, Y, y_bf16, M, N, K, act);
    return;
  }
  dim3 grid((N + 63) / 64, (M + 63) / 64);
  if (x_bf16 && w_bf16)
    gemm_simt_kernel<__nv_bfloat16, __nv_bfloat16><<<grid, 256, 0, st>>>(
        (const __nv_bfloat16*)X, (const __nv_bfloat16*)W, b, Y, y_bf16, M, N, K, act);
  else if (!x_bf16 && !w_bf16)
    gemm_simt_kernel<float, float><<<grid, 256, 0, st>>>((const float*)X, (const float*)W, b, Y, y_bf16, M, N, K, act);
  else if (x_bf16)
    gemm_simt_kernel<__nv_bfloat16, float><<<grid, 256, 0, st>>>((const __nv_bfloat16*)X, (const float*)W, b, Y,
                                                                 y_bf16, M, N, K, act);
  else
    gemm_simt_kernel<float, __nv_bfloat16><<<grid, 256, 0, st>>>((const float*)X, (const __nv_bfloat16*)W, b, Y,
                                                                 y_bf16, M, N, K, act);
  CK(cudaGetLastError());
}

void mlp_small(const void* X, int bf16, const void* const* Ws, const float* const* bs, const int* dims, int L, void* Y,
               int y_bf16, int M, int act, int last_act, cudaStream_t st) {
  if (L > 8) fail(DUET_EUNSUPPORTED, "mlp: at most 8 layers");
  MlpArgs a{};
  int maxd = 0;
  for (int i = 0; i <= L; ++i) {
    a.dims[i] = dims[i];
    maxd = std::max(maxd, dims[i]);
  }
  for (int i = 0; i < L; ++i) {
    a.W[i] = Ws[i];
    a.b[i] = bs[i];
  }
  a.L = L;
  size_t smem = (size_t)2 * 4 * maxd * sizeof(float);
  if (smem > 200 * 1024) fail(DUET_EUNSUPPORTED, "mlp: layer too wide for the fused small-M kernel");
  if (smem > 48 * 1024) CK(cudaFuncSetAttribute(mlp_small_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  launch_pdl(mlp_small_kernel, dim3((M + 3) / 4), dim3(1024), smem, st, X, bf16, a, Y, y_bf16, M, act, last_act, maxd);
  CK(cudaGetLastError());
}

void rnn_step_simt(int kind, const float* gx, const void* Whh, int w_bf16, const float* bhh_n, const void* h_prev,
                   void* h_next, int h_bf16, float* c_state, int M, int H, cudaStream_t st) {
  dim3 grid((H + 31) / 32, (M + 7) / 8);
  if (kind == EPI_LSTM)
    rnn_step_simt_kernel<4><<<grid, 256, 0, st>>>(gx, Whh, w_bf16, bhh_n, h_prev, h_next, h_bf16, c_state, M, H);
  else
    rnn_step_simt_kernel<3><<<grid, 256, 0, st>>>(gx, Whh, w_bf16, bhh_n, h_prev, h_next, h_bf16, c_state, M, H);
  CK(cudaGetLastError());
}

}  // namespace duet
