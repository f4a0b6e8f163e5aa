// MT-DNN shared encoder kernels ("a lexicon encoder and a
// multi-layer bidirectional Transformer encoder", Fig. 3).  The projections (QKV, output, FFN with
// GELU in the epilogue) and the task heads run on the linear-layer GEMMs; what is left here is
// row-wise and latency-bound at the paper's batch of 1:
//   bert_embed     LN(E_tok[tok] + E_pos[s] + E_seg[seg])        one warp per row, registers only
//   add_layernorm  LN(a + b) (post-LN residual)                   one warp per row
//   attention      softmax(Q K^T / sqrt(dh)) V per (sequence, head) with K^T and V staged in
//                  shared memory (fp32), one warp per query row, the S scores spread over lanes
//   select_rows    the [CLS] row of every sequence
#include <cuda_bf16.h>

#include "kernels.h"
#include "ptx.cuh"

namespace duet {

namespace {

constexpr float kLnEps = 1e-12f;  // BERT's LayerNorm epsilon (oracle/forward.py LN_EPS)
constexpr int kMaxV = 32;         // H <= 32 * 32

__device__ __forceinline__ float ldv(const void* p, int64_t i, int bf16) {
  return bf16 ? __bfloat162float(reinterpret_cast<const __nv_bfloat16*>(p)[i]) : reinterpret_cast<const float*>(p)[i];
}
__device__ __forceinline__ void stv(void* p, int64_t i, float v, int bf16) {
  if (bf16)
    reinterpret_cast<__nv_bfloat16*>(p)[i] = __float2bfloat16_rn(v);
  else
    reinterpret_cast<float*>(p)[i] = v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// Row-wise LayerNorm kernels: one warp per row, NV = H / 32 values per lane (compile time; H is a
// multiple of 32 here, other H take the generic NV = 32 path with guards).  gamma / beta are
// loaded with the row, before the two shuffle reductions, so a row costs one memory round trip.
template <typename T>
__device__ __forceinline__ float ldt(const T* p, int64_t i) {
  return to_f(p[i]);
}

template <int NV, typename T>
__device__ __forceinline__ void ln_store(float (&v)[NV], int H, const float (&g)[NV], const float (&be)[NV], T* y,
                                         int64_t row, int lane) {
  constexpr bool kExact = NV < kMaxV;  // H == 32 * NV
  float s = 0.0f;
#pragma unroll
  for (int k = 0; k < NV; ++k)
    if (kExact || lane + 32 * k < H) s += v[k];
  const float mean = warp_sum(s) / (float)H;
  float q = 0.0f;
#pragma unroll
  for (int k = 0; k < NV; ++k)
    if (kExact || lane + 32 * k < H) {
      const float d = v[k] - mean;
      q = fmaf(d, d, q);
    }
  const float rstd = rsqrtf(warp_sum(q) / (float)H + kLnEps);
#pragma unroll
  for (int k = 0; k < NV; ++k) {
    const int i = lane + 32 * k;
    if (kExact || i < H) y[row * H + i] = from_f<T>((v[k] - mean) * rstd * g[k] + be[k]);
  }
}

template <int NV>
__device__ __forceinline__ void ld_gb(const float* g, const float* beta, int H, int lane, float (&gv)[NV],
                                      float (&bv)[NV]) {
#pragma unroll
  for (int k = 0; k < NV; ++k) {
    const int i = lane + 32 * k;
    const bool ok = NV < kMaxV || i < H;
    gv[k] = ok ? __ldg(g + i) : 0.0f;
    bv[k] = ok ? __ldg(beta + i) : 0.0f;
  }
}

template <int NV, typename T>
__global__ void bert_embed_kernel(const int32_t* tok, const int32_t* seg, const T* Etok, const T* Epos,
                                  const T* Eseg, const float* g, const float* beta, T* y, int B, int S, int H) {
  const int row = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  float gv[NV], bv[NV];
  if (row < B * S) ld_gb<NV>(g, beta, H, lane, gv, bv);  // parameters: before the PDL wait
  ptx::pdl_wait();
  ptx::pdl_trigger();
  if (row >= B * S) return;
  const int s = row % S;
  const int64_t t = tok[row], sg = seg[row];
  float v[NV];
#pragma unroll
  for (int k = 0; k < NV; ++k) {
    const int i = lane + 32 * k;
    v[k] = (NV < kMaxV || i < H) ? ldt(Etok, t * H + i) + ldt(Epos, (int64_t)s * H + i) + ldt(Eseg, sg * H + i) : 0.0f;
  }
  ln_store<NV, T>(v, H, gv, bv, y, row, lane);
}

template <int NV, typename T>
__global__ void add_layernorm_kernel(const T* a, const T* b, const float* g, const float* beta, T* y, int64_t rows,
                                     int H) {
  const int64_t row = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  float gv[NV], bv[NV];
  if (row < rows) ld_gb<NV>(g, beta, H, lane, gv, bv);
  ptx::pdl_wait();
  ptx::pdl_trigger();
  if (row >= rows) return;
  float v[NV];
#pragma unroll
  for (int k = 0; k < NV; ++k) {
    const int i = lane + 32 * k;
    v[k] = (NV < kMaxV || i < H) ? ldt(a, row * H + i) + ldt(b, row * H + i) : 0.0f;
  }
  ln_store<NV, T>(v, H, gv, bv, y, row, lane);
}

constexpr int kAttWarps = 8;
constexpr int kAttQ = 8;       // query rows per CTA (1 per warp: B * heads * S warps in flight)
constexpr int kAttMaxT = 16;   // S <= 32 * 16
constexpr int kAttMaxDV = 4;   // dh <= 128

// grid (B * heads, ceil(S / kAttQ)); smem (fp32): K^T [dh][Sp + 1] (padded row: conflict-free
// transposed stores), V [Sp][dh], one dh-vector of Q per warp; Sp = S rounded up to 32 with zero
// keys / values, so the score and PV loops run whole 32-key chunks (padded scores are masked).
// Each lane owns keys lane + 32 t (independent FMA chains over t) and output columns lane + 32 v.
// NT = ceil(S / 32) key chunks and DV = dh / 32 output columns per lane are compile-time: with
// runtime bounds every predicated-off FMA of the 16 x 4 register tiles still issued (4.5x the
// instructions; ncu: issue-bound at 35 us for BERT-base's 12 heads x 128 tokens).
template <int NT, int DV>
__global__ void __launch_bounds__(32 * kAttWarps) attention_kernel(const void* qkv, void* out, int bf16, int S,
                                                                  int heads, int dh) {
  extern __shared__ float att_smem[];
  const int bh = blockIdx.x, b = bh / heads, h = bh % heads;
  const int H = heads * dh, ld = 3 * H;
  constexpr int nt = NT, dv = DV;
  const int Sp = 32 * nt, ldk = Sp + 1;
  float* Kt = att_smem;
  float* Vs = Kt + (size_t)dh * ldk;
  float* Qs = Vs + (size_t)Sp * dh;
  float* Ps = Qs + (size_t)kAttWarps * dh;  // [warps][Sp] softmax probabilities
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  ptx::pdl_wait();
  ptx::pdl_trigger();
  const int64_t base = (int64_t)b * S * ld + (int64_t)h * dh;
  // K / V rows -> smem in 16-byte chunks (8 bf16 / 4 fp32 of one row): every thread issues up to 8
  // independent chunk loads before converting and storing them (ncu: the scalar 2-byte loads of
  // the first version left ~45% of the samples stalled on this phase)
  {
    const int esz = bf16 ? 2 : 4, epc = 16 / esz, cpr = dh / epc, per = Sp * cpr, nch = 2 * per;
    const uint8_t* src = reinterpret_cast<const uint8_t*>(qkv);
    for (int c0 = threadIdx.x; c0 < nch; c0 += 8 * blockDim.x) {
      uint4 raw[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int c = c0 + u * blockDim.x;
        raw[u] = make_uint4(0u, 0u, 0u, 0u);
        if (c < nch) {
          const int kvs = c / per, rem = c - kvs * per, j = rem / cpr, d0 = (rem - j * cpr) * epc;
          if (j < S)
            raw[u] = __ldg(reinterpret_cast<const uint4*>(src + (base + (int64_t)j * ld + (1 + kvs) * H + d0) * esz));
        }
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int c = c0 + u * blockDim.x;
        if (c >= nch) break;
        const int kvs = c / per, rem = c - kvs * per, j = rem / cpr, d0 = (rem - j * cpr) * epc;
        float f[8];
        if (bf16) {
          const __nv_bfloat16* hv = reinterpret_cast<const __nv_bfloat16*>(&raw[u]);
#pragma unroll
          for (int i = 0; i < 8; ++i) f[i] = __bfloat162float(hv[i]);
        } else {
          f[0] = __uint_as_float(raw[u].x), f[1] = __uint_as_float(raw[u].y);
          f[2] = __uint_as_float(raw[u].z), f[3] = __uint_as_float(raw[u].w);
        }
        if (kvs == 0) {
          for (int i = 0; i < epc; ++i) Kt[(d0 + i) * ldk + j] = f[i];
        } else {
          for (int i = 0; i < epc; ++i) Vs[j * dh + d0 + i] = f[i];
        }
      }
    }
  }
  __syncthreads();
  const float scale = rsqrtf((float)dh);
  float* q = Qs + warp * dh;
  for (int qi = blockIdx.y * kAttQ + warp; qi < min(S, (int)(blockIdx.y + 1) * kAttQ); qi += kAttWarps) {
    for (int d = lane; d < dh; d += 32) q[d] = ldv(qkv, base + (int64_t)qi * ld + d, bf16) * scale;
    __syncwarp();
    float p[NT];
#pragma unroll
    for (int t = 0; t < NT; ++t) p[t] = 0.0f;
#pragma unroll 4
    for (int d = 0; d < dh; ++d) {
      const float qd = q[d];
      const float* kr = Kt + d * ldk + lane;
#pragma unroll
      for (int t = 0; t < NT; ++t) p[t] = fmaf(qd, kr[32 * t], p[t]);
    }
    float m = -INFINITY;
#pragma unroll
    for (int t = 0; t < NT; ++t)
      if (t * 32 + lane < S) m = fmaxf(m, p[t]);
    m = warp_max(m);
    float sum = 0.0f;
#pragma unroll
    for (int t = 0; t < NT; ++t) {
      p[t] = (t * 32 + lane < S) ? expf(p[t] - m) : 0.0f;
      sum += p[t];
    }
    const float inv = 1.0f / warp_sum(sum);
    // probabilities -> this warp's smem row, then every lane walks the keys with broadcast reads
    // (a shuffle per key serialised the PV loop on its latency)
    float* pw = Ps + warp * Sp;
#pragma unroll
    for (int t = 0; t < NT; ++t) pw[t * 32 + lane] = p[t];
    __syncwarp();
    float acc[4][DV];
#pragma unroll
    for (int v = 0; v < DV; ++v) acc[0][v] = acc[1][v] = acc[2][v] = acc[3][v] = 0.0f;
    const float* vr = Vs + lane;
#pragma unroll 8
    for (int jj = 0; jj < 32 * NT; ++jj) {
      const float pj = pw[jj];
#pragma unroll
      for (int v = 0; v < DV; ++v) acc[jj & 3][v] = fmaf(pj, vr[jj * dh + 32 * v], acc[jj & 3][v]);
    }
#pragma unroll
    for (int v = 0; v < DV; ++v) acc[0][v] += acc[1][v] + acc[2][v] + acc[3][v];
    const int64_t o = ((int64_t)b * S + qi) * H + (int64_t)h * dh + lane;
#pragma unroll
    for (int v = 0; v < DV; ++v) stv(out, o + 32 * v, acc[0][v] * inv, bf16);
    __syncwarp();
  }
}

template <typename T>
__global__ void select_rows_kernel(const T* x, T* y, int64_t rows, int64_t cols, int64_t stride, int64_t offset) {
  ptx::pdl_wait();
  ptx::pdl_trigger();
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < rows * cols; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = e / cols, c = e - r * cols;
    y[e] = x[(offset + r * stride) * cols + c];
  }
}

int att_nt(int S) {  // key chunks of the instantiated kernel (1, 2, 4, 6, 8, 12, 16)
  const int nt = (S + 31) / 32;
  return nt <= 2 ? nt : nt <= 4 ? 4 : nt <= 6 ? 6 : nt <= 8 ? 8 : nt <= 12 ? 12 : 16;
}
size_t att_smem_bytes(int S, int dh) {
  const size_t sp = (size_t)32 * att_nt(S);
  return ((size_t)dh * (sp + 1) + sp * dh + (size_t)kAttWarps * dh + (size_t)kAttWarps * sp) * 4;
}

}  // namespace

// NV = H / 32 when H is one of the compiled multiples of 32, else the guarded NV = 32 path
#define DUET_LN_NV(H, X) \
  switch (H) {           \
    case 128: X(4)       \
    case 256: X(8)       \
    case 512: X(16)      \
    case 768: X(24)      \
    case 1024: X(32)     \
    default: X(kMaxV)    \
  }

void bert_embed(const int32_t* tok, const int32_t* seg, const void* Etok, const void* Epos, const void* Eseg,
                const float* g, const float* beta, void* y, int bf16, int B, int S, int H, int64_t V, cudaStream_t st) {
  (void)V;
  if (H > 32 * kMaxV) fail(DUET_EUNSUPPORTED, "bert_embed: hidden size > 1024");
  const int rows = B * S, wpb = 4;
  const dim3 grid((rows + wpb - 1) / wpb), block(32 * wpb);
#define X(NV)                                                                                                   \
  if (bf16)                                                                                                     \
    return launch_pdl(bert_embed_kernel<NV, __nv_bfloat16>, grid, block, 0, st, tok, seg,                       \
                      (const __nv_bfloat16*)Etok, (const __nv_bfloat16*)Epos, (const __nv_bfloat16*)Eseg, g, beta, \
                      (__nv_bfloat16*)y, B, S, H);                                                              \
  return launch_pdl(bert_embed_kernel<NV, float>, grid, block, 0, st, tok, seg, (const float*)Etok,              \
                    (const float*)Epos, (const float*)Eseg, g, beta, (float*)y, B, S, H);
  DUET_LN_NV(H, X)
#undef X
}

void add_layernorm(const void* a, const void* b, const float* g, const float* beta, void* y, int bf16, int64_t rows,
                   int H, cudaStream_t st) {
  if (H > 32 * kMaxV) fail(DUET_EUNSUPPORTED, "add_layernorm: hidden size > 1024");
  const int wpb = 4;
  const dim3 grid((unsigned)((rows + wpb - 1) / wpb)), block(32 * wpb);
#define X(NV)                                                                                                  \
  if (bf16)                                                                                                    \
    return launch_pdl(add_layernorm_kernel<NV, __nv_bfloat16>, grid, block, 0, st, (const __nv_bfloat16*)a,    \
                      (const __nv_bfloat16*)b, g, beta, (__nv_bfloat16*)y, rows, H);                           \
  return launch_pdl(add_layernorm_kernel<NV, float>, grid, block, 0, st, (const float*)a, (const float*)b, g,   \
                    beta, (float*)y, rows, H);
  DUET_LN_NV(H, X)
#undef X
}
#undef DUET_LN_NV

bool attention_ok(int S, int dh) {
  return S >= 1 && S <= 32 * kAttMaxT && (dh == 32 || dh == 64 || dh == 128) && att_smem_bytes(S, dh) <= 227 * 1024;
}

template <int NT>
void launch_attention(int dv, const void* qkv, void* out, int bf16, int B, int S, int heads, int dh, size_t smem,
                      cudaStream_t st) {
  const dim3 grid(B * heads, (S + kAttQ - 1) / kAttQ), block(32 * kAttWarps);
  auto go = [&](auto kern) {
    static size_t attr = 0;  // one per instantiation
    if (smem > 48 * 1024 && smem > attr) {
      CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      attr = smem;
    }
    launch_pdl(kern, grid, block, smem, st, qkv, out, bf16, S, heads, dh);
  };
  if (dv == 1) return go(attention_kernel<NT, 1>);
  if (dv == 2) return go(attention_kernel<NT, 2>);
  return go(attention_kernel<NT, 4>);
}

void attention(const void* qkv, void* out, int bf16, int B, int S, int heads, int dh, cudaStream_t st) {
  if (!attention_ok(S, dh)) fail(DUET_EUNSUPPORTED, "attention: needs S <= 512, dh in {32, 64, 128} and K, V in 227 KB of smem");
  const size_t smem = att_smem_bytes(S, dh);
  const int dv = dh / 32;
  switch (att_nt(S)) {
    case 1: return launch_attention<1>(dv, qkv, out, bf16, B, S, heads, dh, smem, st);
    case 2: return launch_attention<2>(dv, qkv, out, bf16, B, S, heads, dh, smem, st);
    case 4: return launch_attention<4>(dv, qkv, out, bf16, B, S, heads, dh, smem, st);
    case 6: return launch_attention<6>(dv, qkv, out, bf16, B, S, heads, dh, smem, st);
    case 8: return launch_attention<8>(dv, qkv, out, bf16, B, S, heads, dh, smem, st);
    case 12: return launch_attention<12>(dv, qkv, out, bf16, B, S, heads, dh, smem, st);
    default: return launch_attention<16>(dv, qkv, out, bf16, B, S, heads, dh, smem, st);
  }
}

void select_rows(const void* x, void* y, int esize, int64_t rows, int64_t cols, int64_t stride, int64_t offset,
                 cudaStream_t st) {
  const int64_t n = rows * cols;
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, 4096);
  if (esize == 2)
    launch_pdl(select_rows_kernel<uint16_t>, dim3(grid), dim3(256), 0, st, (const uint16_t*)x, (uint16_t*)y, rows,
               cols, stride, offset);
  else if (esize == 4)
    launch_pdl(select_rows_kernel<uint32_t>, dim3(grid), dim3(256), 0, st, (const uint32_t*)x, (uint32_t*)y, rows,
               cols, stride, offset);
  else
    fail(DUET_EUNSUPPORTED, "select_rows: element size must be 2 or 4");
}

}  // namespace duet
