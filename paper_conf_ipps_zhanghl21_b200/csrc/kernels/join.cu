// Branch joins, elementwise ops and pooling.  Joins are one warp per row
// with a shuffle reduction (coalesced lane-strided reads of each branch's row).
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

__device__ __forceinline__ int row_of_warp() { return blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); }

__global__ void reduce_sum_kernel(const void* x, int bf16, const float* b, float* y, int B, int K) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  int row = row_of_warp(), lane = threadIdx.x & 31;
  if (row >= B) return;
  float s = 0.0f;
  for (int k = lane; k < K; k += 32) s += ldx(x, (int64_t)row * K + k, bf16);
  s = warp_sum(s);
  if (lane == 0) y[row] = s + b[0];
}

__global__ void dot_join_kernel(const float* s, const void* a, int bf16, const float* w, const float* b, float* y,
                                int B, int K) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  int row = row_of_warp(), lane = threadIdx.x & 31;
  if (row >= B) return;
  float acc = 0.0f;
  for (int k = lane; k < K; k += 32) acc = fmaf(ldx(a, (int64_t)row * K + k, bf16), w[k], acc);
  acc = warp_sum(acc);
  if (lane == 0) y[row] = sigmoidf_acc(s[row] + acc + b[0]);
}

__global__ void cosine_join_kernel(const void* a, const void* b, int bf16, float* y, int B, int K) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  int row = row_of_warp(), lane = threadIdx.x & 31;
  if (row >= B) return;
  float ab = 0.0f, aa = 0.0f, bb = 0.0f;
  for (int k = lane; k < K; k += 32) {
    float x = ldx(a, (int64_t)row * K + k, bf16), z = ldx(b, (int64_t)row * K + k, bf16);
    ab = fmaf(x, z, ab);
    aa = fmaf(x, x, aa);
    bb = fmaf(z, z, bb);
  }
  ab = warp_sum(ab);
  aa = warp_sum(aa);
  bb = warp_sum(bb);
  if (lane == 0) {
    float den = sqrtf(aa) * sqrtf(bb);
    y[row] = den > 0.0f ? ab / den : 0.0f;
  }
}

struct HeadArgs {
  const void* p[8];
  int K[8];
  int bf16[8];
  int n;
};

__global__ void concat_head_kernel(HeadArgs h, const float* w, const float* b, float* y, int B, int act) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  int row = row_of_warp(), lane = threadIdx.x & 31;
  if (row >= B) return;
  float acc = 0.0f;
  int off = 0;
  for (int i = 0; i < h.n; ++i) {
    for (int k = lane; k < h.K[i]; k += 32) acc = fmaf(ldx(h.p[i], (int64_t)row * h.K[i] + k, h.bf16[i]), w[off + k], acc);
    off += h.K[i];
  }
  acc = warp_sum(acc);
  if (lane == 0) y[row] = apply_act(acc + b[0], act);
}

struct LogitArgs {
  const float* p[16];
  int n;
};

__global__ void logit_join_kernel(LogitArgs a, float* y, int B, int mean) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  int row = blockIdx.x * blockDim.x + threadIdx.x;
  if (row >= B) return;
  float s = 0.0f;
  for (int i = 0; i < a.n; ++i) s += a.p[i][row];
  if (mean) s /= (float)a.n;
  y[row] = sigmoidf_acc(s);
}

template <typename T>
__global__ void add_act_kernel(const T* a, const T* b, T* y, int64_t n, int act) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    y[i] = from_f<T>(apply_act(to_f(a[i]) + to_f(b[i]), act));
}

template <typename T>
__global__ void sigmoid_kernel(const T* x, T* y, int64_t n) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    y[i] = from_f<T>(sigmoidf_acc(to_f(x[i])));
}

template <typename T>
__global__ void maxpool_kernel(const T* x, T* y, int N, int H, int W, int C, int k, int s, int p, int Ho, int Wo) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  int64_t total = (int64_t)N * Ho * Wo * C;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    int c = (int)(i % C);
    int64_t t = i / C;
    int wo = (int)(t % Wo);
    t /= Wo;
    int ho = (int)(t % Ho);
    int n = (int)(t / Ho);
    float m = -INFINITY;
    for (int r = 0; r < k; ++r) {
      int hi = ho * s - p + r;
      if (hi < 0 || hi >= H) continue;
      for (int q = 0; q < k; ++q) {
        int wi = wo * s - p + q;
        if (wi < 0 || wi >= W) continue;
        m = fmaxf(m, to_f(x[(((int64_t)n * H + hi) * W + wi) * C + c]));
      }
    }
    y[i] = from_f<T>(m);
  }
}

// global average pool: one thread per (n, c), coalesced over c
template <typename T>
__global__ void avgpool_kernel(const T* x, T* y, int N, int HW, int C) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  int64_t total = (int64_t)N * C;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    int c = (int)(i % C);
    int64_t n = i / C;
    float s = 0.0f;
    const T* base = x + n * HW * C + c;
    for (int j = 0; j < HW; ++j) s += to_f(base[(int64_t)j * C]);
    y[i] = from_f<T>(s / (float)HW);
  }
}

// global average pool for small maps (HW < 8, e.g. c5's 1x1 layer-4 output), NHWC bf16, C % 8 == 0:
// one thread per (image, 8-channel chunk), 16-byte loads, the HW positions summed in order in fp32
// (the same order as avgpool_kernel; the scalar kernel took 16 us for c5's 4 MB)
__global__ void avgpool_small8_kernel(const uint4* __restrict__ x, uint4* __restrict__ y, int N, int HW, int C8) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  const int total = N * C8;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < total; i += gridDim.x * blockDim.x) {
    const int n = i / C8, c8 = i - n * C8;
    float acc[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) acc[e] = 0.0f;
    for (int j = 0; j < HW; ++j) {
      const uint4 v = __ldg(x + ((size_t)n * HW + j) * C8 + c8);
      const __nv_bfloat16* b = reinterpret_cast<const __nv_bfloat16*>(&v);
#pragma unroll
      for (int e = 0; e < 8; ++e) acc[e] += __bfloat162float(b[e]);
    }
    uint4 o;
    __nv_bfloat16* ob = reinterpret_cast<__nv_bfloat16*>(&o);
#pragma unroll
    for (int e = 0; e < 8; ++e) ob[e] = __float2bfloat16_rn(acc[e] / (float)HW);
    y[i] = o;
  }
}

int warp_rows_grid(int B) { return (B + 7) / 8; }

// NHWC bf16 maxpool, 8 channels (16 B) per thread, 32-bit index math (C % 8 == 0)
__global__ void maxpool8_kernel(const uint4* __restrict__ x, uint4* __restrict__ y, int N, int H, int W, int C8, int k,
                                int s, int p, int Ho, int Wo) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  const int total = N * Ho * Wo * C8;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < total; i += gridDim.x * blockDim.x) {
    int c8 = i % C8;
    int t = i / C8;
    int wo = t % Wo;
    t /= Wo;
    int ho = t % Ho;
    int n = t / Ho;
    float m[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) m[e] = -INFINITY;
    for (int r = 0; r < k; ++r) {
      int hi = ho * s - p + r;
      if (hi < 0 || hi >= H) continue;
      for (int q = 0; q < k; ++q) {
        int wi = wo * s - p + q;
        if (wi < 0 || wi >= W) continue;
        uint4 v = __ldg(x + ((n * H + hi) * W + wi) * C8 + c8);
        const __nv_bfloat16* b = reinterpret_cast<const __nv_bfloat16*>(&v);
#pragma unroll
        for (int e = 0; e < 8; ++e) m[e] = fmaxf(m[e], __bfloat162float(b[e]));
      }
    }
    uint4 o;
    __nv_bfloat16* ob = reinterpret_cast<__nv_bfloat16*>(&o);
#pragma unroll
    for (int e = 0; e < 8; ++e) ob[e] = __float2bfloat16_rn(m[e]);
    y[i] = o;
  }
}

// ResNet maxpool (3x3, stride 2, pad 1) on NHWC bf16, 8 channels (16 B) per thread: the nine
// window loads are unrolled and issued together (clamped addresses, out-of-window taps masked to
// -inf), so each thread keeps nine 16-B requests in flight instead of one per loop trip.
__global__ void maxpool3s2_kernel(const uint4* __restrict__ x, uint4* __restrict__ y, int N, int H, int W, int C8,
                                  int Ho, int Wo) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  const int total = N * Ho * Wo * C8;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < total; i += gridDim.x * blockDim.x) {
    const int c8 = i % C8;
    int t = i / C8;
    const int wo = t % Wo;
    t /= Wo;
    const int ho = t % Ho;
    const int n = t / Ho;
    uint4 v[9];
    bool ok[9];
#pragma unroll
    for (int r = 0; r < 3; ++r)
#pragma unroll
      for (int q = 0; q < 3; ++q) {
        const int hi = 2 * ho - 1 + r, wi = 2 * wo - 1 + q;
        ok[r * 3 + q] = hi >= 0 && hi < H && wi >= 0 && wi < W;
        const int hc = min(max(hi, 0), H - 1), wc = min(max(wi, 0), W - 1);
        v[r * 3 + q] = __ldg(x + ((n * H + hc) * W + wc) * C8 + c8);
      }
    float m[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) m[e] = -INFINITY;
#pragma unroll
    for (int j = 0; j < 9; ++j) {
      const __nv_bfloat16* b = reinterpret_cast<const __nv_bfloat16*>(&v[j]);
#pragma unroll
      for (int e = 0; e < 8; ++e) m[e] = ok[j] ? fmaxf(m[e], __bfloat162float(b[e])) : m[e];
    }
    uint4 o;
    __nv_bfloat16* ob = reinterpret_cast<__nv_bfloat16*>(&o);
#pragma unroll
    for (int e = 0; e < 8; ++e) ob[e] = __float2bfloat16_rn(m[e]);
    y[i] = o;
  }
}

// ResNet maxpool (3x3, stride 2, pad 1), NHWC bf16, C % 8 == 0, staged (round 2): a CTA pools
// output rows [ho0, ho0 + k) of one image from the input rows they read, [2 ho0 - 1, 2 ho0 + 2k),
// which are contiguous in NHWC: ONE bulk copy into shared memory, then the nine taps per 16-byte
// output chunk come from there (the per-thread nine-load kernel above reached ~0.5 of HBM).  Every
// window holds its centre pixel, so the max starts from it (no -inf padding needed).
__device__ __forceinline__ uint4 bmax8(uint4 a, uint4 b) {
  uint32_t* pa = reinterpret_cast<uint32_t*>(&a);
  const uint32_t* pb = reinterpret_cast<const uint32_t*>(&b);
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    __nv_bfloat162 r = __hmax2(*reinterpret_cast<const __nv_bfloat162*>(&pa[q]), *reinterpret_cast<const __nv_bfloat162*>(&pb[q]));
    pa[q] = *reinterpret_cast<uint32_t*>(&r);
  }
  return a;
}
__global__ void maxpool3s2_rows_kernel(const uint4* __restrict__ x, uint4* __restrict__ y, int H, int W, int C8, int Ho,
                                       int Wo, int k) {
  extern __shared__ __align__(128) uint4 srows[];
  __shared__ __align__(8) uint64_t bar;
  const int bands = (Ho + k - 1) / k;
  const int n = blockIdx.x / bands, ho0 = (blockIdx.x % bands) * k, ho1 = min(Ho, ho0 + k);
  const int r0 = max(0, 2 * ho0 - 1), r1 = min(H, 2 * ho1);
  const uint32_t bytes = (uint32_t)((r1 - r0) * W * C8 * 16);
  if (threadIdx.x == 0) {
    ptx::mbar_init(&bar, 1);
    ptx::fence_mbar_init();
  }
  __syncthreads();
  ptx::pdl_wait();
  ptx::pdl_trigger();
  if (threadIdx.x == 0) {
    ptx::mbar_arrive_expect_tx(&bar, bytes);
    ptx::bulk_g2s(srows, x + ((size_t)n * H + r0) * W * C8, bytes, &bar);
  }
  ptx::mbar_wait(&bar, 0);
  const int total = (ho1 - ho0) * Wo * C8;
  uint4* yo = y + ((size_t)n * Ho + ho0) * Wo * C8;
  for (int i = threadIdx.x; i < total; i += blockDim.x) {
    const int c8 = i % C8, t = i / C8, wo = t % Wo, ho = ho0 + t / Wo;
    uint4 m = srows[((2 * ho - r0) * W + 2 * wo) * C8 + c8];
#pragma unroll
    for (int r = -1; r <= 1; ++r) {
      const int hi = 2 * ho + r;
      if (hi < r0 || hi >= r1) continue;
#pragma unroll
      for (int q = -1; q <= 1; ++q) {
        const int wi = 2 * wo + q;
        if (wi < 0 || wi >= W || (r == 0 && q == 0)) continue;
        m = bmax8(m, srows[((hi - r0) * W + wi) * C8 + c8]);
      }
    }
    yo[i] = m;
  }
}

// global average pool, NHWC bf16, C % 8 == 0: block = (image n, 32 chunks of 8 channels); its 8
// warps split the HW positions (warp w takes j = w, w + 8, ...), lane = channel chunk, 4 loads in
// flight per lane, then the 8 partial sums are added in warp order in shared memory (fixed order:
// deterministic).
__global__ void avgpool8_kernel(const uint4* __restrict__ x, uint4* __restrict__ y, int HW, int C8) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  __shared__ float part[8][32][8];
  const int n = blockIdx.x;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int c8 = blockIdx.y * 32 + lane;
  float acc[8];
#pragma unroll
  for (int e = 0; e < 8; ++e) acc[e] = 0.0f;
  if (c8 < C8) {
    const uint4* base = x + (size_t)n * HW * C8 + c8;
    int j = warp;
    for (; j + 24 < HW; j += 32) {
      uint4 v[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) v[u] = __ldg(base + (size_t)(j + 8 * u) * C8);
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const __nv_bfloat16* b = reinterpret_cast<const __nv_bfloat16*>(&v[u]);
#pragma unroll
        for (int e = 0; e < 8; ++e) acc[e] += __bfloat162float(b[e]);
      }
    }
    for (; j < HW; j += 8) {
      const uint4 v = __ldg(base + (size_t)j * C8);
      const __nv_bfloat16* b = reinterpret_cast<const __nv_bfloat16*>(&v);
#pragma unroll
      for (int e = 0; e < 8; ++e) acc[e] += __bfloat162float(b[e]);
    }
  }
#pragma unroll
  for (int e = 0; e < 8; ++e) part[warp][lane][e] = acc[e];
  __syncthreads();
  if (warp == 0 && c8 < C8) {
    float s[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) {
      s[e] = 0.0f;
#pragma unroll
      for (int w = 0; w < 8; ++w) s[e] += part[w][lane][e];
    }
    uint4 o;
    __nv_bfloat16* ob = reinterpret_cast<__nv_bfloat16*>(&o);
    const float inv = 1.0f / (float)HW;
#pragma unroll
    for (int e = 0; e < 8; ++e) ob[e] = __float2bfloat16_rn(s[e] * inv);
    y[(size_t)n * C8 + c8] = o;
  }
}

}  // namespace

void reduce_sum(const void* x, int x_bf16, const float* b, float* y, int B, int K, cudaStream_t st) {
  if (!B) return;
  launch_pdl(reduce_sum_kernel, dim3(warp_rows_grid(B)), dim3(256), 0, st, x, x_bf16, b, y, B, K);
  CK(cudaGetLastError());
}

void dot_join(const float* s, const void* a, int a_bf16, const float* w, const float* b, float* y, int B, int K,
              cudaStream_t st) {
  if (!B) return;
  launch_pdl(dot_join_kernel, dim3(warp_rows_grid(B)), dim3(256), 0, st, s, a, a_bf16, w, b, y, B, K);
  CK(cudaGetLastError());
}

void cosine_join(const void* a, const void* b, int bf16, float* y, int B, int K, cudaStream_t st) {
  if (!B) return;
  launch_pdl(cosine_join_kernel, dim3(warp_rows_grid(B)), dim3(256), 0, st, a, b, bf16, y, B, K);
  CK(cudaGetLastError());
}

void concat_head(const void* const* parts, const int* Ks, const int* bf16s, int n, const float* w, const float* b,
                 float* y, int B, int act, cudaStream_t st) {
  if (n > 8) fail(DUET_EUNSUPPORTED, "concat_head: at most 8 parts");
  HeadArgs h{};
  for (int i = 0; i < n; ++i) {
    h.p[i] = parts[i];
    h.K[i] = Ks[i];
    h.bf16[i] = bf16s[i];
  }
  h.n = n;
  if (!B) return;
  launch_pdl(concat_head_kernel, dim3(warp_rows_grid(B)), dim3(256), 0, st, h, w, b, y, B, act);
  CK(cudaGetLastError());
}

void logit_join(const float* const* parts, int n, float* y, int B, int mean, cudaStream_t st) {
  if (n > 16) fail(DUET_EUNSUPPORTED, "logit join: at most 16 branches");
  LogitArgs a{};
  for (int i = 0; i < n; ++i) a.p[i] = parts[i];
  a.n = n;
  if (!B) return;
  launch_pdl(logit_join_kernel, dim3((B + 255) / 256), dim3(256), 0, st, a, y, B, mean);
  CK(cudaGetLastError());
}

void add_act(const void* a, const void* b, void* y, int bf16, int64_t n, int act, cudaStream_t st) {
  if (!n) return;
  if (bf16)
    launch_pdl(add_act_kernel<__nv_bfloat16>, dim3(grid_for(n, 256)), dim3(256), 0, st, (const __nv_bfloat16*)a, (const __nv_bfloat16*)b,
                                                                  (__nv_bfloat16*)y, n, act);
  else
    launch_pdl(add_act_kernel<float>, dim3(grid_for(n, 256)), dim3(256), 0, st, (const float*)a, (const float*)b, (float*)y, n, act);
  CK(cudaGetLastError());
}

void sigmoid_ew(const void* x, void* y, int bf16, int64_t n, cudaStream_t st) {
  if (!n) return;
  if (bf16)
    launch_pdl(sigmoid_kernel<__nv_bfloat16>, dim3(grid_for(n, 256)), dim3(256), 0, st, (const __nv_bfloat16*)x, (__nv_bfloat16*)y, n);
  else
    launch_pdl(sigmoid_kernel<float>, dim3(grid_for(n, 256)), dim3(256), 0, st, (const float*)x, (float*)y, n);
  CK(cudaGetLastError());
}

void maxpool_nhwc(const void* x, void* y, int bf16, int N, int H, int W, int C, int k, int s, int p, int Ho, int Wo,
                  cudaStream_t st) {
  int64_t total = (int64_t)N * Ho * Wo * C;
  if (!total) return;
  const bool vec = bf16 && C % 8 == 0 && total / 8 < INT32_MAX && (int64_t)N * H * W * C / 8 < INT32_MAX &&
                   ((uintptr_t)x % 16) == 0 && ((uintptr_t)y % 16) == 0;
  const int64_t row_bytes = (int64_t)W * C * 2;
  if (vec && k == 3 && s == 2 && p == 1 && 3 * row_bytes <= 64 * 1024) {
    // output rows per CTA: the most whose input rows fit in 64 KB of shared memory
    const int kr = std::max(1, std::min(Ho, (int)((64 * 1024 / row_bytes - 1) / 2)));
    const int bands = (Ho + kr - 1) / kr;
    const size_t smem = (size_t)std::min<int64_t>(H, 2 * kr + 1) * row_bytes;
    static size_t attr = 0;
    if (smem > attr) {
      CK(cudaFuncSetAttribute(maxpool3s2_rows_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      attr = smem;
    }
    launch_plain(maxpool3s2_rows_kernel, dim3((unsigned)((int64_t)N * bands)), dim3(256), smem, st, (const uint4*)x,
                 (uint4*)y, H, W, C / 8, Ho, Wo, kr);
    CK(cudaGetLastError());
    return;
  }
  if (vec && k == 3 && s == 2 && p == 1) {
    launch_plain(maxpool3s2_kernel, dim3(grid_for(total / 8, 256, 16)), dim3(256), 0, st, (const uint4*)x, (uint4*)y, N, H,
                 W, C / 8, Ho, Wo);
    CK(cudaGetLastError());
    return;
  }
  if (vec) {
    launch_plain(maxpool8_kernel, dim3(grid_for(total / 8, 256, 16)), dim3(256), 0, st, (const uint4*)x, (uint4*)y, N, H, W,
               C / 8, k, s, p, Ho, Wo);
    CK(cudaGetLastError());
    return;
  }
  if (bf16)
    launch_plain(maxpool_kernel<__nv_bfloat16>, dim3(grid_for(total, 256)), dim3(256), 0, st, (const __nv_bfloat16*)x, (__nv_bfloat16*)y, N,
                                                                       H, W, C, k, s, p, Ho, Wo);
  else
    launch_plain(maxpool_kernel<float>, dim3(grid_for(total, 256)), dim3(256), 0, st, (const float*)x, (float*)y, N, H, W, C, k, s, p, Ho,
                                                               Wo);
  CK(cudaGetLastError());
}

void avgpool_nhwc(const void* x, void* y, int bf16, int N, int H, int W, int C, cudaStream_t st) {
  int64_t total = (int64_t)N * C;
  if (!total) return;
  if (bf16 && C % 8 == 0 && H * W >= 8 && ((uintptr_t)x % 16) == 0 && ((uintptr_t)y % 16) == 0) {
    launch_plain(avgpool8_kernel, dim3(N, (C / 8 + 31) / 32), dim3(256), 0, st, (const uint4*)x, (uint4*)y, H * W, C / 8);
    CK(cudaGetLastError());
    return;
  }
  if (bf16 && C % 8 == 0 && total / 8 < INT32_MAX && ((uintptr_t)x % 16) == 0 && ((uintptr_t)y % 16) == 0) {
    launch_plain(avgpool_small8_kernel, dim3(grid_for(total / 8, 256)), dim3(256), 0, st, (const uint4*)x, (uint4*)y, N,
                 H * W, C / 8);
    CK(cudaGetLastError());
    return;
  }
  if (bf16)
    launch_plain(avgpool_kernel<__nv_bfloat16>, dim3(grid_for(total, 256)), dim3(256), 0, st, (const __nv_bfloat16*)x, (__nv_bfloat16*)y, N,
                                                                       H * W, C);
  else
    launch_plain(avgpool_kernel<float>, dim3(grid_for(total, 256)), dim3(256), 0, st, (const float*)x, (float*)y, N, H * W, C);
  CK(cudaGetLastError());
}

}  // namespace duet
