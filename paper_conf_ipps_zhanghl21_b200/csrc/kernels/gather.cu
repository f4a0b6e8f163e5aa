// Embedding gathers: feature hashing, wide gather-reduce, deep
// gather-concat, token embedding.  HBM-bound: each thread moves 16-byte vectors with
// non-allocating loads (the table is read once per lookup, never reused by this kernel), stores
// are coalesced (consecutive threads write consecutive 16 B of the concat buffer), and several
// independent lookups per thread are in flight (grid-stride x4 unroll).
#include <cuda_bf16.h>

#include "kernels.h"
#include "ptx.cuh"

namespace duet {

int num_sms(int device) {
  static int cache[64] = {0};
  if (device < 0 || device >= 64) device = 0;
  if (!cache[device]) {
    int v = 0;
    CK(cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, device));
    cache[device] = v;
  }
  return cache[device];
}

namespace {

__device__ __forceinline__ uint4 ld_stream16(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

// id = x mod V (floor modulo)
__device__ __forceinline__ int32_t hash_id(int64_t x, int64_t V) {
  int64_t r;
  if ((uint64_t)x < (1ULL << 32) && V < (1LL << 32))
    r = (int64_t)((uint32_t)x % (uint32_t)V);  // 32-bit path (the recipe's raw ids are < 2^31)
  else {
    r = x % V;
    if (r < 0) r += V;
  }
  return (int32_t)r;
}

// A gather's ids (the hash node's int32 output), read through the read-only path.
struct IdSrc {
  const int32_t* ids;
  __device__ __forceinline__ int32_t operator()(int64_t i) const { return __ldg(ids + i); }
};

__global__ void hash_mod_kernel(const int64_t* __restrict__ raw, int32_t* __restrict__ ids, int64_t n, int64_t V) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    ids[i] = hash_id(raw[i], V);
}

template <typename T>
__global__ void gather_sum_kernel(const IdSrc ids, const T* __restrict__ tab,
                                  const float* __restrict__ b, float* __restrict__ y, int B, int F, int64_t R) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  const int warps = (blockDim.x >> 5);
  const int row = blockIdx.x * warps + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (row >= B) return;
  float acc = 0.0f;
  for (int f = lane; f < F; f += 32) {
    int id = ids((int64_t)row * F + f);
    acc += to_f(tab[(size_t)f * R + id]);
  }
  acc = warp_sum(acc);
  if (lane == 0) y[row] = acc + __ldg(b);
}

// out row r (of `rows`) <- table row src_row(r); vpr 16-byte vectors per row.
template <int MODE>  // 0: gather_concat (row r = b*F + f), 1: embed_seq (row r = t*B + b)
__global__ void gather_rows16_kernel(const IdSrc idx, const uint8_t* __restrict__ tab,
                                     uint8_t* __restrict__ out, int64_t rows, int vpr, int64_t row_bytes, int F,
                                     int64_t R, int B, int S) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  const int64_t total = rows * vpr;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  for (; v < total; v += 4 * stride) {
    uint4 val[4];
    int64_t dst[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      int64_t vv = v + u * stride;
      dst[u] = -1;
      if (vv < total) {
        int64_t r = vv / vpr;
        int k = (int)(vv - r * vpr);
        int64_t trow;
        if (MODE == 0) {
          int f = (int)(r % F);
          trow = (int64_t)f * R + idx(r);
        } else {
          int64_t t = r / B;
          int64_t b = r - t * B;
          trow = idx(b * S + t);
        }
        val[u] = ld_stream16(tab + trow * row_bytes + (int64_t)k * 16);
        dst[u] = r * row_bytes + (int64_t)k * 16;
      }
    }
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (dst[u] >= 0) *reinterpret_cast<uint4*>(out + dst[u]) = val[u];
  }
}

// Same with a power-of-two number of 16-byte vectors per row and 32-bit index math (the generic
// kernel's 64-bit divisions per vector dominated its issue time): VPR lanes per row, four rows in
// flight per thread.
template <int MODE, int VPR, int UNR = 4>
__global__ void __launch_bounds__(256) gather_rows16p2_kernel(const IdSrc idx,
                                                              const uint8_t* __restrict__ tab,
                                                              uint8_t* __restrict__ out, int rows, int F,
                                                              int64_t R, int B, int S) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  constexpr int RB = VPR * 16;
  const int k = threadIdx.x & (VPR - 1);
  const int rows_per_pass = (int)(gridDim.x * blockDim.x) / VPR;
  for (int r0 = (int)(blockIdx.x * blockDim.x + threadIdx.x) / VPR; r0 < rows; r0 += UNR * rows_per_pass) {
    uint4 val[UNR];
#pragma unroll
    for (int u = 0; u < UNR; ++u) {
      const int r = r0 + u * rows_per_pass;
      if (r < rows) {
        int64_t trow;
        if (MODE == 0) {
          trow = (int64_t)(r % F) * R + idx(r);
        } else {
          const int t = r / B, b = r - t * B;
          trow = idx((int64_t)b * S + t);
        }
        val[u] = ld_stream16(tab + trow * RB + k * 16);
      }
    }
#pragma unroll
    for (int u = 0; u < UNR; ++u) {
      const int r = r0 + u * rows_per_pass;
      if (r < rows) *reinterpret_cast<uint4*>(out + (int64_t)r * RB + k * 16) = val[u];
    }
  }
}

template <int MODE>
__global__ void gather_rows_bytes_kernel(const IdSrc idx, const uint8_t* __restrict__ tab,
                                         uint8_t* __restrict__ out, int64_t rows, int64_t row_bytes, int F,
                                         int64_t R, int B, int S) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  const int64_t total = rows * row_bytes;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < total; v += (int64_t)gridDim.x * blockDim.x) {
    int64_t r = v / row_bytes;
    int64_t k = v - r * row_bytes;
    int64_t trow;
    if (MODE == 0) {
      trow = (int64_t)(r % F) * R + idx(r);
    } else {
      int64_t t = r / B, b = r - t * B;
      trow = idx(b * S + t);
    }
    out[v] = tab[trow * row_bytes + k];
  }
}

__device__ __forceinline__ uint32_t mix32(uint32_t x) {
  x ^= x >> 16;
  x *= 0x7feb352du;
  x ^= x >> 15;
  x *= 0x846ca68bu;
  x ^= x >> 16;
  return x;
}

__global__ void fill_random_kernel(void* p, int dtype, int64_t n, int64_t high, uint64_t seed) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint32_t h = mix32((uint32_t)i ^ mix32((uint32_t)seed ^ (uint32_t)(i >> 32)));
    switch (dtype) {
      case kI64: reinterpret_cast<int64_t*>(p)[i] = (int64_t)(h & 0x7fffffffu); break;
      case kI32: reinterpret_cast<int32_t*>(p)[i] = (int32_t)(h % (uint32_t)(high > 0 ? high : 1)); break;
      case kF32: reinterpret_cast<float*>(p)[i] = (float)(h >> 8) * (2.0f / 16777216.0f) - 1.0f; break;
      case kBF16:
        reinterpret_cast<__nv_bfloat16*>(p)[i] = __float2bfloat16((float)(h >> 8) * (2.0f / 16777216.0f) - 1.0f);
        break;
    }
  }
}

__global__ void permute_rows_kernel(const uint32_t* __restrict__ src, uint32_t* __restrict__ dst,
                                    const int32_t* __restrict__ map, int64_t rows, int64_t words) {
  const int64_t total = rows * words;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < total; v += (int64_t)gridDim.x * blockDim.x) {
    int64_t r = v / words, k = v - r * words;
    int32_t s = map[r];
    dst[v] = s >= 0 ? src[(int64_t)s * words + k] : 0u;
  }
}


}  // namespace

int grid_for(int64_t work, int threads, int per_sm) {
  int64_t g = (work + threads - 1) / threads;
  int dev = 0;
  cudaGetDevice(&dev);
  int64_t cap = (int64_t)num_sms(dev) * per_sm;
  if (g > cap) g = cap;
  if (g < 1) g = 1;
  return (int)g;
}

void hash_mod(const int64_t* raw, int32_t* ids, int64_t n, int64_t V, cudaStream_t st) {
  if (n == 0) return;
  launch_pdl(hash_mod_kernel, dim3(grid_for(n, 256)), dim3(256), 0, st, raw, ids, n, V);
  CK(cudaGetLastError());
}

void gather_sum(const int32_t* ids_, const void* T, int t_bf16, const float* b, float* y, int B, int F, int64_t R,
                cudaStream_t st) {
  if (B == 0) return;
  const IdSrc ids{ids_};
  int blocks = (B + 7) / 8;
  if (t_bf16)
    launch_pdl(gather_sum_kernel<__nv_bfloat16>, dim3(blocks), dim3(256), 0, st, ids, (const __nv_bfloat16*)T, b, y, B, F, R);
  else
    launch_pdl(gather_sum_kernel<float>, dim3(blocks), dim3(256), 0, st, ids, (const float*)T, b, y, B, F, R);
  CK(cudaGetLastError());
}

static void gather_rows(int mode, const IdSrc idx, const void* tab, int esize, void* out, int64_t rows, int D,
                        int F, int64_t R, int B, int S, cudaStream_t st) {
  if (rows == 0) return;
  int64_t rb = (int64_t)D * esize;
  bool vec = (rb % 16 == 0) && ((uintptr_t)tab % 16 == 0) && ((uintptr_t)out % 16 == 0);
  const int vpr16 = (int)(rb / 16);
  if (vec && rows < (1LL << 30) && (vpr16 == 4 || vpr16 == 8 || vpr16 == 16 || vpr16 == 32)) {
    // (8 rows in flight per thread measured slower than 4 at every c3-c5 embedding shape)
    const int g = grid_for((rows * vpr16 + 3) / 4, 256, 16);
#define DUET_G16(M, V)                                                                                             \
  if (mode == M && vpr16 == V)                                                                                     \
    launch_pdl(gather_rows16p2_kernel<M, V>, dim3(g), dim3(256), 0, st, idx, (const uint8_t*)tab, (uint8_t*)out,  \
               (int)rows, F, R, B, S);
    // 512-byte rows (E = 256 bf16: c3-c5's token embeddings) took the generic kernel's 64-bit
    // divisions until round 2: c5's b2_x 32.8 -> 16.1 us
    DUET_G16(0, 4) DUET_G16(0, 8) DUET_G16(0, 16) DUET_G16(0, 32) DUET_G16(1, 4) DUET_G16(1, 8) DUET_G16(1, 16)
    DUET_G16(1, 32)
#undef DUET_G16
  } else if (vec) {
    int vpr = (int)(rb / 16);
    int64_t total = rows * vpr;
    int g = grid_for((total + 3) / 4, 256, 16);
    if (mode == 0)
      launch_pdl(gather_rows16_kernel<0>, dim3(g), dim3(256), 0, st, idx, (const uint8_t*)tab, (uint8_t*)out, rows, vpr, rb, F, R, B, S);
    else
      launch_pdl(gather_rows16_kernel<1>, dim3(g), dim3(256), 0, st, idx, (const uint8_t*)tab, (uint8_t*)out, rows, vpr, rb, F, R, B, S);
  } else {
    int g = grid_for(rows * rb, 256);
    if (mode == 0)
      launch_pdl(gather_rows_bytes_kernel<0>, dim3(g), dim3(256), 0, st, idx, (const uint8_t*)tab, (uint8_t*)out, rows, rb, F, R, B, S);
    else
      launch_pdl(gather_rows_bytes_kernel<1>, dim3(g), dim3(256), 0, st, idx, (const uint8_t*)tab, (uint8_t*)out, rows, rb, F, R, B, S);
  }
  CK(cudaGetLastError());
}

void gather_concat(const int32_t* ids, const void* E, int esize, void* X, int B, int F, int64_t R, int D,
                   cudaStream_t st) {
  gather_rows(0, IdSrc{ids}, E, esize, X, (int64_t)B * F, D, F, R, B, 0, st);
}

void embed_seq(const int32_t* tok, const void* E, int esize, void* X, int B, int S, int64_t V, int D,
               cudaStream_t st) {
  gather_rows(1, IdSrc{tok}, E, esize, X, (int64_t)B * S, D, 1, V, B, S, st);
}

void fill_random(void* p, int dtype, int64_t n, int64_t high, uint64_t seed, cudaStream_t st) {
  if (n == 0) return;
  fill_random_kernel<<<grid_for(n, 256), 256, 0, st>>>(p, dtype, n, high, seed);
  CK(cudaGetLastError());
}

void permute_rows(const void* src, void* dst, const int32_t* map, int64_t rows_dst, int64_t row_bytes,
                  cudaStream_t st) {
  if (row_bytes % 4) fail(DUET_EUNSUPPORTED, "permute_rows: row bytes must be a multiple of 4");
  int64_t words = row_bytes / 4;
  if (rows_dst * words == 0) return;
  permute_rows_kernel<<<grid_for(rows_dst * words, 256), 256, 0, st>>>((const uint32_t*)src, (uint32_t*)dst, map,
                                                                       rows_dst, words);
  CK(cudaGetLastError());
}

}  // namespace duet
