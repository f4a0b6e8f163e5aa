// Direct tcgen05 kernel for small-channel convolutions (ResNet's 7x7/2 stem over 3 channels).
//
// The C % 64 == 0 layers use im2col-mode TMA (conv_tc.cu); with C = 3 a tap is 6 bytes, far below
// TMA's 16-byte minimum, and the explicit im2col buffer (M x 152 bf16 = 244 MB at batch 64) made the
// stem HBM-bound at ~0.5 ms.  Here the im2col happens in shared memory instead:
//
//   tile   = rp consecutive output rows of one image (rp = 128 / Wo: one row at 224x224, eight at
//            32x32): rp * Wo <= 128 pixels = the UMMA M rows (the rest stay zero)
//   patch  = the (rp-1)*stride + kh input rows that tile reads: nbx TMA boxes of [rows x 256 elements] whose
//            starts are STEP = 256 - 24 elements apart, so every pixel's 24-element window lies
//            inside one box (3 requests per tile for the stem; TMA's per-request cost, not bytes,
//            bounded a row-per-request version).  Out-of-image rows / columns, including the
//            padding, are zero-filled by TMA.
//   A tile = built by 4 builder warps from the patch: K is ordered (kh, then a 24-element segment
//            holding [d dummy][kw*C window elements][zeros]) so that every 16-byte K chunk of a row
//            is four aligned 4-byte words of one patch row; written in the SWIZZLE_128B K-major
//            layout the UMMA descriptor expects
//   W      = [Co, 192] in the same K order (packed once at build), TMA-loaded once, resident
//   MMA    = one thread, UMMA 128 x Co x 16, accumulator double-buffered in TMEM
//   epilogue = 4 warps: bias (folded BN) + activation, bf16, the tile's Wo x Co outputs are
//            contiguous in NHWC
//
// Persistent: grid = min(tiles, SMs); patch, A and TMEM are double-buffered so the TMA of tile
// i+2, the build of i+1, the MMAs of i and the epilogue of i-1 overlap.
#include "../common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace duet {

namespace {

constexpr int SEG = 24;             // K elements per kernel row (kh)
constexpr int KPAD = 192;           // K padded to three 64-element SWIZZLE_128B atoms
constexpr int ATOMS = KPAD / 64;
constexpr int ROWS = 128;           // UMMA M
constexpr int A_ATOM_BYTES = ROWS * 128;
constexpr int A_BYTES = ATOMS * A_ATOM_BYTES;  // 48 KB
constexpr int NB = 8;               // builder warps (two threads per output pixel, kh rows split)
constexpr int NE = 4;               // epilogue warps
constexpr int PW = NB + 1 + NE;     // patch producer warp (tile fetch + patch TMA), last
constexpr int THREADS = 32 * (PW + 1);
constexpr int NPMAX = 8;            // max patch buffers
constexpr int BOXW = 256;           // patch box width (elements)
constexpr int STEP = BOXW - SEG;    // element distance between consecutive boxes

__host__ __device__ constexpr int tmem_cols(int co) {
  return 2 * co <= 32 ? 32 : 2 * co <= 64 ? 64 : 2 * co <= 128 ? 128 : 256;
}

struct StemGeom {
  int N, H, W, C, Co, kh, kw, stride, pad, Ho, Wo;
  int L;       // PA: left padding in elements rounded up to 8 (box starts are 16-byte aligned)
  int d;       // dummy elements at the start of each segment (aligns the window to 4 bytes)
  int rowb;    // bytes per box row = BOXW * 2
  int bw, nbx; // box width (BOXW) and boxes per tile
  int ksteps;  // UMMA K steps (16) covering kh * SEG
  int rp;      // output rows per tile
  int bh;      // patch box rows = (rp - 1) * stride + kh
  int tpi;     // tiles per image = ceil(Ho / rp)
  int np;      // patch buffers in flight (prefetch depth; HBM latency is the bound with 2)
  int act;
  int dbg;     // micro-benchmark switches (DUET_STEM_DBG): 1 skip build, 2 skip MMA, 4 skip stores,
               // 8 skip patch TMA (builders use stale patches)
  unsigned* ctr;  // [2] dynamic tile counter + exit count (null: static tiles block + i grid)
};

__global__ void stem_pack_kernel(const __nv_bfloat16* __restrict__ wf, int64_t ldw, __nv_bfloat16* __restrict__ wk,
                                 int Co, int kh, int kw, int C, int d) {
  const int co = blockIdx.x;
  for (int k = threadIdx.x; k < KPAD; k += blockDim.x) {
    const int r = k / SEG, j = k % SEG - d;
    __nv_bfloat16 v = __float2bfloat16(0.0f);
    if (r < kh && j >= 0 && j < kw * C) v = wf[(int64_t)co * ldw + (int64_t)r * kw * C + j];
    wk[(int64_t)co * KPAD + k] = v;
  }
}

template <int CO>
__global__ void __launch_bounds__(THREADS, 1)
    conv_stem_kernel(const __grid_constant__ CUtensorMap tmX, const __grid_constant__ CUtensorMap tmW,
                     const float* __restrict__ bias, __nv_bfloat16* __restrict__ y, const StemGeom g) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;                                  // 2 x A_BYTES
  uint8_t* sW = sA + 2 * A_BYTES;                      // ATOMS x CO x 128 B
  uint8_t* sP = sW + ATOMS * CO * 128;                 // np x nbx x kh x rowb
  const int bbytes = g.bh * g.rowb;                    // one box
  const int pbytes = g.nbx * bbytes;
  uint64_t* bars = reinterpret_cast<uint64_t*>(sP + g.np * pbytes);
  uint64_t* patch_full = bars;          // [np] TMA tx
  uint64_t* a_full = bars + NPMAX;      // [2] builders -> MMA
  uint64_t* a_empty = a_full + 2;       // [2] MMA commit -> builders
  uint64_t* t_full = a_full + 4;        // [2] MMA commit -> epilogue
  uint64_t* t_empty = a_full + 6;       // [2] epilogue -> MMA
  uint64_t* w_full = a_full + 8;
  uint64_t* patch_empty = a_full + 9;   // [np] builders -> patch producer
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(patch_empty + NPMAX);
  float* s_bias = reinterpret_cast<float*>(patch_empty + NPMAX + 1);
  // tile of local work item i: s_tile[i % 16] (-1 = no more work), written by the patch issuer,
  // published through ring_full[i % 16]; the MMA warp and the epilogue each read it and arrive on
  // ring_empty[i % 16] before the slot is reused
  __shared__ int s_tile[16];
  __shared__ uint64_t ring_full[16], ring_empty[16];

  const int warp = ptx::warp_id();
  const int lane = threadIdx.x & 31;
  const int tiles = g.N * g.tpi;
  const uint32_t patch_tx = (uint32_t)pbytes;

  if (threadIdx.x == 0) {
    ptx::tma_prefetch(&tmX);
    ptx::tma_prefetch(&tmW);
    for (int i = 0; i < g.np; ++i) {
      ptx::mbar_init(&patch_full[i], 1);
      ptx::mbar_init(&patch_empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(&a_full[i], 1);
      ptx::mbar_init(&a_empty[i], 1);
      ptx::mbar_init(&t_full[i], 1);
      ptx::mbar_init(&t_empty[i], NE);
    }
    ptx::mbar_init(w_full, 1);
    for (int i = 0; i < 16; ++i) {
      ptx::mbar_init(&ring_full[i], 1);
      ptx::mbar_init(&ring_empty[i], 2);
    }
    ptx::fence_mbar_init();
  }
  // zero both A tiles (rows >= Wo and K >= kh*SEG stay zero for good)
  for (int i = threadIdx.x; i < (2 * A_BYTES) / 16; i += THREADS) reinterpret_cast<uint4*>(sA)[i] = make_uint4(0, 0, 0, 0);
  for (int i = threadIdx.x; i < CO; i += THREADS) s_bias[i] = bias[i];
  ptx::fence_async_smem();
  __syncthreads();
  if (threadIdx.x == 0) {  // weights: graph parameters, loaded before the PDL wait
    ptx::mbar_arrive_expect_tx(w_full, ATOMS * CO * 128);
    for (int a = 0; a < ATOMS; ++a) ptx::tma_load_2d(&tmW, w_full, sW + a * CO * 128, a * 64, 0);
  }
  ptx::pdl_wait();  // before TMEM is taken
  if (warp == NB) {
    ptx::tmem_alloc(tmem_slot, tmem_cols(CO));
    ptx::tmem_relinquish();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  ptx::pdl_trigger();

  // Dynamic tile scheduling when g.ctr is set (a CTA whose SM frees up early keeps taking tiles;
  // see conv_tc.cu): item i's tile is fetched when its patch is issued.  A -1 item still arrives on
  // patch_full (no TMA) so the builders, then the MMA warp, then the epilogue see the end.
  auto issue_patch = [&](int i) {  // TMA of local item i's input rows into patch buffer i % np
    int tile = g.ctr ? (int)atomicAdd(g.ctr, 1u) : (int)(blockIdx.x + i * gridDim.x);
    if (tile >= tiles) {
      tile = -1;
      if (g.ctr && atomicAdd(g.ctr + 1, 1u) == gridDim.x - 1) {  // last CTA done fetching: reset
        g.ctr[0] = 0;
        g.ctr[1] = 0;
      }
    }
    if (i >= 16) ptx::mbar_wait(&ring_empty[i & 15], (uint32_t)(((i >> 4) - 1) & 1));
    s_tile[i & 15] = tile;
    ptx::mbar_arrive(&ring_full[i & 15]);
    const int pb = i % g.np;
    if (tile < 0 || (g.dbg & 8)) {
      ptx::mbar_arrive(&patch_full[pb]);
      return;
    }
    const int n = tile / g.tpi, ho = (tile % g.tpi) * g.rp;
    uint8_t* dst = sP + pb * pbytes;
    ptx::mbar_arrive_expect_tx(&patch_full[pb], patch_tx);
    for (int b = 0; b < g.nbx; ++b)
      ptx::tma_load_3d(&tmX, &patch_full[pb], dst + b * bbytes, b * STEP - g.L, ho * g.stride - g.pad, n);
  };

  if (warp == PW) {
    // ---------------- patch producer: tile fetch + patch TMA, np items ahead of the builders ----------------
    // (its own warp since round 2: issued by builder thread 0, the tile counter's atomic round trip
    // sat on the builders' critical path -- c4 stem 114 -> 88 us, c5 133 -> 104 us, CUDA-graph timing)
    if (lane == 0) {
      for (int i = 0;; ++i) {
        if (i >= g.np) ptx::mbar_wait(&patch_empty[i % g.np], (uint32_t)(((i / g.np) - 1) & 1));
        issue_patch(i);
        if (s_tile[i & 15] < 0) break;
      }
    }
  } else if (warp < NB) {
    // ---------------- builders: patch -> A (im2col in shared memory) ----------------
    const int m = threadIdx.x & (ROWS - 1);  // output pixel (UMMA row) of this thread
    const int rr = m / g.Wo, wo = m % g.Wo;   // output row within the tile, column
    const int kh_half = (g.kh + 1) / 2;
    const int r0 = threadIdx.x < ROWS ? 0 : kh_half, r1 = threadIdx.x < ROWS ? kh_half : g.kh;
    // this pixel's window: box b, element offset o (even: 4-byte aligned words), box row rr*stride
    const int off = g.stride * g.C * wo + g.L - g.pad * g.C - g.d;
    const int src0 = (off / STEP) * bbytes + (off % STEP) * 2 + rr * g.stride * g.rowb;
    const bool live_px = m < g.rp * g.Wo;
    for (int i = 0;; ++i) {
      const int p = i & 1, pb = i % g.np;
      ptx::mbar_wait(&patch_full[pb], (i / g.np) & 1);
      if (i >= 2) ptx::mbar_wait(&a_empty[p], ((i >> 1) - 1) & 1);
      if (s_tile[i & 15] < 0) break;  // (visible: the issuer wrote it before arriving on patch_full)
      if (live_px && !(g.dbg & 1)) {
        const uint8_t* prow = sP + pb * pbytes + src0;
        uint8_t* arow = sA + p * A_BYTES + m * 128;
#pragma unroll 4
        for (int r = r0; r < r1; ++r) {
          const uint32_t* s32 = reinterpret_cast<const uint32_t*>(prow + r * (BOXW * 2));
#pragma unroll
          for (int s = 0; s < 3; ++s) {
            const uint4 v = make_uint4(s32[4 * s], s32[4 * s + 1], s32[4 * s + 2], s32[4 * s + 3]);
            const int c = r * 3 + s;  // 16-byte K chunk
            *reinterpret_cast<uint4*>(arow + (c >> 3) * A_ATOM_BYTES + (((c & 7) ^ (m & 7)) << 4)) = v;
          }
        }
      }
      ptx::fence_async_smem();
      asm volatile("bar.sync 2, %0;" ::"n"(32 * NB) : "memory");  // A[p] built, patch[p] consumed
      if (threadIdx.x == 0) {
        ptx::mbar_arrive(&a_full[p]);
        ptx::mbar_arrive(&patch_empty[pb]);
      }
    }
  } else if (warp == NB) {
    // ---------------- MMA issuer ----------------
    // the whole warp walks the loop (uniform descriptors); elect.sync issues each UMMA
    {
      constexpr uint32_t idesc = ptx::idesc_bf16(ROWS, CO);
      ptx::mbar_wait(w_full, 0);
      const uint64_t da0 = ptx::desc_sw128(ptx::smem_u32(sA));
      const uint64_t dw0 = ptx::desc_sw128(ptx::smem_u32(sW));
      for (int i = 0;; ++i) {
        const int b = i & 1;
        ptx::mbar_wait(&ring_full[i & 15], (uint32_t)((i >> 4) & 1));
        const int tile = s_tile[i & 15];
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(&ring_empty[i & 15]);
        if (tile < 0) break;
        ptx::mbar_wait(&a_full[b], (i >> 1) & 1);
        if (i >= 2) ptx::mbar_wait(&t_empty[b], ((i >> 1) - 1) & 1);
        ptx::tc_fence_after();
        const uint64_t da = da0 + (uint64_t)((b * A_BYTES) >> 4);
        for (int k = 0; k < ((g.dbg & 2) ? 0 : g.ksteps); ++k) {
          const int atom = k >> 2, kk = k & 3;
          ptx::umma_bf16_elect(tmem + b * CO, da + (uint64_t)((atom * A_ATOM_BYTES + kk * 32) >> 4),
                               dw0 + (uint64_t)((atom * CO * 128 + kk * 32) >> 4), idesc, k != 0);
        }
        ptx::umma_commit_elect(&a_empty[b]);
        ptx::umma_commit_elect(&t_full[b]);
      }
    }
  } else {
    // ---------------- epilogue ----------------
    const int q = warp & 3;  // TMEM lane quarter of this warp
    const int m = q * 32 + lane;
    for (int i = 0;; ++i) {
      const int b = i & 1;
      ptx::mbar_wait(&ring_full[i & 15], (uint32_t)((i >> 4) & 1));
      const int tile = s_tile[i & 15];
      asm volatile("bar.sync 3, %0;" ::"n"(32 * NE) : "memory");  // every epilogue thread has read it
      if (threadIdx.x == 32 * (NB + 1)) ptx::mbar_arrive(&ring_empty[i & 15]);
      if (tile < 0) break;
      ptx::mbar_wait(&t_full[b], (i >> 1) & 1);
      ptx::tc_fence_after();
      float v[CO];
      const uint32_t tq = tmem + b * CO + ((uint32_t)(q * 32) << 16);
      if constexpr (CO % 64 == 0) {
#pragma unroll
        for (int c = 0; c < CO; c += 64) ptx::tmem_ld64(tq + c, v + c);
      } else {
#pragma unroll
        for (int c = 0; c < CO; c += 16) ptx::tmem_ld16(tq + c, v + c);
      }
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&t_empty[b]);
      const int n = tile / g.tpi, ho0 = (tile % g.tpi) * g.rp;
      if (m < g.rp * g.Wo && ho0 + m / g.Wo < g.Ho && !(g.dbg & 4)) {
        // the tile's rows are consecutive in NHWC: pixel m of the tile is pixel m after (n, ho0, 0)
        __nv_bfloat16* out = y + (((int64_t)n * g.Ho + ho0) * g.Wo + m) * CO;
#pragma unroll
        for (int c = 0; c < CO; c += 16) {
          float t[16];
#pragma unroll
          for (int u = 0; u < 16; ++u) t[u] = v[c + u];
          bias_act<16>(t, s_bias + c, g.act);
          store_row16(out + c, t);
        }
      }
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == NB) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, tmem_cols(CO));
  }
}

StemGeom geom(const ConvShape& s, int act) {
  StemGeom g{s.N, s.H, s.W, s.C, s.Co, s.kh, s.kw, s.stride, s.pad, s.Ho, s.Wo, 0, 0, 0, 0, 0, 0, 0, 0, 0, 2, act, 0};
  g.rp = std::max(1, std::min(ROWS / std::max(1, s.Wo), s.Ho));
  g.bh = (g.rp - 1) * s.stride + s.kh;
  g.tpi = (s.Ho + g.rp - 1) / g.rp;
  g.dbg = getenv("DUET_STEM_DBG") ? atoi(getenv("DUET_STEM_DBG")) : 0;
  g.d = (s.pad * s.C) & 1;
  g.L = (s.pad * s.C + g.d + 7) / 8 * 8;
  g.rowb = BOXW * 2;
  g.bw = BOXW;
  // pixel m's window starts `off(m) = stride*C*m + L - pad*C - d` elements after box 0's start;
  // box b starts at image element b*STEP - L (a multiple of 8) and holds windows with
  // off / STEP == b
  g.nbx = (s.stride * s.C * (s.Wo - 1) + g.L - s.pad * s.C - g.d) / STEP + 1;
  g.ksteps = (s.kh * SEG + 15) / 16;
  const size_t fixed = 1024 + 2 * A_BYTES + (size_t)ATOMS * s.Co * 128 + (2 * NPMAX + 10) * 8 + (size_t)s.Co * 4;
  const size_t pb = (size_t)g.nbx * g.bh * g.rowb;
  g.np = (int)std::min<size_t>(NPMAX, (227 * 1024 - 512 - fixed) / pb);  // 512: the static tile ring
  if (g.np < 2) g.np = 2;  // (conv_stem_ok rejects shapes that do not fit two)
  return g;
}

size_t stem_smem(const StemGeom& g) {
  return 1024 + 2 * A_BYTES + (size_t)ATOMS * g.Co * 128 + (size_t)g.np * g.nbx * g.bh * g.rowb +
         (2 * NPMAX + 10) * 8 + (size_t)g.Co * 4;
}

}  // namespace

bool conv_stem_ok(const ConvShape& s) {
  if (s.kh > KPAD / SEG || s.Wo > ROWS || s.Co % 16 || s.Co < 16 || s.Co > 128) return false;
  if ((std::min(ROWS / std::max(1, s.Wo), s.Ho) - 1) * s.stride + s.kh > 256) return false;  // TMA box rows
  if ((s.pad * s.C) % 2 + s.kw * s.C > SEG) return false;      // window fits a segment
  if ((s.stride * s.C) % 2) return false;                        // 4-byte aligned windows
  if ((s.W * s.C) % 8) return false;                             // TMA row pitch (16 B)
  return stem_smem(geom(s, 0)) + 512 <= 227 * 1024;  // + the static tile ring
}

void conv_stem_pack(const void* wf, int64_t ldw, void* wk, const ConvShape& s, cudaStream_t st) {
  const int d = (s.pad * s.C) & 1;
  stem_pack_kernel<<<s.Co, 64, 0, st>>>((const __nv_bfloat16*)wf, ldw, (__nv_bfloat16*)wk, s.Co, s.kh, s.kw, s.C, d);
  CK(cudaGetLastError());
}

CUtensorMap conv_stem_wmap(const void* wk, int Co) {
  return make_tmap_bf16_2d(wk, Co, KPAD, Co);  // box = 64 K x Co rows, SWIZZLE_128B
}

void conv_stem(const CUtensorMap& tw, const void* x, const float* bias, void* y, const ConvShape& s, int act,
               unsigned* ctr, cudaStream_t st) {
  StemGeom g = geom(s, act);
  g.ctr = ctr;
  CUtensorMap tx;
  cuuint64_t dims[3] = {(cuuint64_t)s.W * s.C, (cuuint64_t)s.H, (cuuint64_t)s.N};
  cuuint64_t strides[2] = {(cuuint64_t)s.W * s.C * 2, (cuuint64_t)s.H * s.W * s.C * 2};
  cuuint32_t box[3] = {(cuuint32_t)BOXW, (cuuint32_t)g.bh, 1};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = tmap_encode_tiled()(&tx, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<void*>(x), dims, strides, box,
                                   estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) fail(DUET_ECUDA, "conv_stem: image tensor map (" + std::to_string((int)r) + ")");
  const size_t smem = stem_smem(g);
  const int tiles = s.N * g.tpi;
  int dev = 0;
  CK(cudaGetDevice(&dev));
  const int grid = std::min(tiles, num_sms(dev));
#define DUET_STEM(COV)                                                                           \
  case COV: {                                                                                    \
    auto kern = conv_stem_kernel<COV>;                                                           \
    static size_t attr = 0;                                                                      \
    if (smem > attr) {                                                                           \
      CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));    \
      attr = smem;                                                                               \
    }                                                                                            \
    launch_pdl_if(pdl_on(true), kern, dim3(grid), dim3(THREADS), smem, st, tx, tw, bias,         \
                  (__nv_bfloat16*)y, g);                                                         \
    return;                                                                                      \
  }
  switch (s.Co) {
    DUET_STEM(16)
    DUET_STEM(32)
    DUET_STEM(48)
    DUET_STEM(64)
    DUET_STEM(80)
    DUET_STEM(96)
    DUET_STEM(112)
    DUET_STEM(128)
  }
#undef DUET_STEM
  fail(DUET_EUNSUPPORTED, "conv_stem: Co must be a multiple of 16 in [16, 128]");
}

}  // namespace duet
