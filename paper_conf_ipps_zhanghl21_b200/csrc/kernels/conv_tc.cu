// Implicit-GEMM convolution on tcgen05 (R-27).
//
//   out[m, co] = act( sum_k A[m, k] * Wf[co, k] + bias[co] (+ res[m, co]) )
//   m = (n, ho, wo) output pixel (NHWC), k = (r, s, c) filter tap x input channel
//
//
// The A operand (im2col) is never materialised: one thread issues, per 64-wide k-block, an
// im2col-mode TMA that gathers 128 consecutive output pixels x 64 channels of filter tap (r, s)
// (padding halo zero-filled by the TMA unit) straight into the SWIZZLE_128B K-major layout UMMA
// reads, plus a tiled TMA of the BN-folded weights [Co, K].  Persistent CTAs walk the tiles with a
// continuous stage ring (2 k-blocks per stage) and a double-buffered TMEM accumulator; 4 epilogue
// warps add the folded BN bias and the optional residual, apply ReLU and store bf16 NHWC.
// Layers with C % 64 != 0 (the 3-channel stem) use im2col_kernel + the CTA-pair GEMM instead.
//
// Tap rectangle (round 2): filter taps whose window lies in the zero padding for EVERY output pixel
// are skipped (their products are exact zeros).  A 3x3 / pad 1 conv on a 1x1 map (c5's ResNet
// layer 4 at 32x32 input) keeps only the centre tap: K drops 9x (57 -> 24 us).  (A split-K variant
// for the under-filled layer-3/4 grids -- fp32 partial tiles + last-arriver reduction -- was built
// and measured slower at every ResNet shape, 1.1-3x.)
#include <cudaTypedefs.h>

#include "../common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace duet {

namespace {

constexpr int CBM = 128;
constexpr int CBK = 64;                 // one SWIZZLE_128B atom of K

// OCC CTAs per SM: the stage ring is split between them (two CTAs hide each other's TMA round
// trips on the 64-channel layers, whose 4-stage ring holds less than one tile)
template <int BN, int OCC = 1, int KB_ = 2>
struct ConvCfg {
  static constexpr int KB = KB_;  // k-blocks per pipeline stage (2 halves the barrier round trips)
  static constexpr int CA_BYTES = KB * CBM * CBK * 2;
  static constexpr int B_ATOM = BN * CBK * 2;
  static constexpr int B_BYTES = KB * B_ATOM;
  static constexpr int STAGE = CA_BYTES + B_BYTES;
  static constexpr int STAGES = (192 * 1024 / OCC) / STAGE > 8 ? 8 : (192 * 1024 / OCC) / STAGE;
  static constexpr int LAG = STAGES - 1;  // cp.async groups kept in flight per producer thread
  static constexpr int TMEM_COLS = BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : 256;  // x2 (double buffer)
  static constexpr int SMEM = STAGES * STAGE + 1024 + 512 + BN * 4;
};

struct ConvArgs {
  const __nv_bfloat16* x;
  const float* bias;
  const __nv_bfloat16* res;
  __nv_bfloat16* y;
  ConvShape s;
  int K;   // kh * kw * C (true reduction length; also the first fully out-of-bounds weight column)
  int act;
  int nkb;             // effective 64-wide k-blocks: taps in the rectangle x C / 64
  int r0, s0, ns;      // tap rectangle: rows r0.., columns s0 .. s0 + ns - 1
  unsigned* ctr;       // [2] dynamic tile counter + exit count (zero between launches; the last
                       // CTA to finish fetching resets both), or null: static tile = block + j grid
  int dbg;             // 1: one producer thread issues A and W (comparisons; DUET_CONV_ISS=1)
};

// TMA-im2col variant (C % 64 == 0): one thread streams both operands; A tile = 128 consecutive
// output pixels x 64 channels of filter tap (r, s) loaded by one im2col TMA.
// ISS2 (round 2): the weights of each stage are issued by their own warp (warp 6, a third reader of the
// tile ring): one thread's copies complete in issue order, and the producer issued an im2col A box
// and a W box per k-block (the same finding)
template <int OCC>
constexpr bool conv_iss2() { return OCC <= 2; }  // three CTAs per SM: 224 threads would cap registers
template <int OCC>
constexpr int conv_threads() { return conv_iss2<OCC>() ? 224 : 192; }

template <int BN, int OCC, int KB>
__global__ void __launch_bounds__(conv_threads<OCC>(), OCC) conv_tma_kernel(const __grid_constant__ CUtensorMap tmX,
                                                            const __grid_constant__ CUtensorMap tmW, const ConvArgs a) {
  using C = ConvCfg<BN, OCC, KB>;
  constexpr int CA_BYTES = C::CA_BYTES;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::STAGES * CA_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(sB + C::STAGES * C::B_BYTES);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tmem_full = empty + C::STAGES;
  uint64_t* tmem_empty = tmem_full + 2;
  uint64_t* tile_full = tmem_empty + 2;   // [4] producer -> MMA / epilogue: s_tile[slot] is set
  uint64_t* tile_empty = tile_full + 4;   // [4] MMA + epilogue have read it
  int* s_tile = reinterpret_cast<int*>(tile_empty + 4);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(s_tile + 4);
  float* s_bias = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(full) + 512);

  const ConvShape& s = a.s;
  const int warp = ptx::warp_id();
  const int lane = threadIdx.x & 31;
  const int64_t M = (int64_t)s.N * s.Ho * s.Wo;
  const int tiles_n = (s.Co + BN - 1) / BN;
  const int64_t n_tiles = ((M + CBM - 1) / CBM) * tiles_n;
  const int cb = s.C / 64;
  const int nk = (a.nkb + KB - 1) / KB;

  if (threadIdx.x == 0) {
    ptx::tma_prefetch(&tmX);
    ptx::tma_prefetch(&tmW);
    for (int i = 0; i < C::STAGES; ++i) {
      ptx::mbar_init(&full[i], (conv_iss2<OCC>() && !(a.dbg & 1)) ? 2 : 1);  // A producer (+ W issuer)
      ptx::mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(&tmem_full[i], 1);
      ptx::mbar_init(&tmem_empty[i], 128);
    }
    for (int i = 0; i < 4; ++i) {
      ptx::mbar_init(&tile_full[i], 1);
      ptx::mbar_init(&tile_empty[i], (conv_iss2<OCC>() && !(a.dbg & 1)) ? 3 : 2);  // MMA, epilogue (+ W issuer)
    }
    ptx::fence_mbar_init();
  }
  // wait for the previous kernel BEFORE taking tensor memory: a PDL-dependent CTA that holds TMEM
  // while it waits can starve a co-resident kernel of another stream (observed as a hang with
  // two slots)
  ptx::pdl_wait();
  if (warp == 1) {
    ptx::tmem_alloc(tmem_slot, 2 * C::TMEM_COLS);
    ptx::tmem_relinquish();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  ptx::pdl_trigger();

  // Tiles are handed out dynamically when a.ctr is set: a CTA that finds its SM free early (the
  // other stream slot's persistent recurrence holds most SMs) keeps taking
  // tiles instead of owning a fixed share that waits for the late CTAs' SMs.  The producer fetches
  // tile j into s_tile[j % 4]; the MMA warp and the epilogue read it from there.
  const bool iss2 = conv_iss2<OCC>() && !(a.dbg & 1);
  if (warp == 0) {
    if (lane == 0) {
      int64_t g = 0;
      for (int j = 0;; ++j) {
        int64_t u = a.ctr ? (int64_t)atomicAdd(a.ctr, 1u) : (int64_t)blockIdx.x + (int64_t)j * gridDim.x;
        const int slot = j & 3;
        if (j >= 4) ptx::mbar_wait(&tile_empty[slot], (uint32_t)(((j >> 2) - 1) & 1));
        s_tile[slot] = u < n_tiles ? (int)u : -1;
        ptx::mbar_arrive(&tile_full[slot]);
        if (u >= n_tiles) {
          // the last CTA to stop fetching resets the counters for the next launch
          if (a.ctr && atomicAdd(a.ctr + 1, 1u) == gridDim.x - 1) {
            a.ctr[0] = 0;
            a.ctr[1] = 0;
          }
          break;
        }
        const int64_t tile = u;
        const int n0 = (int)(tile % tiles_n) * BN;
        const int64_t m0 = (tile / tiles_n) * CBM;
        const int wo = (int)(m0 % s.Wo);
        const int64_t q0 = m0 / s.Wo;
        const int ho = (int)(q0 % s.Ho);
        const int nn = (int)(q0 / s.Ho);
        const int wb = wo * s.stride - s.pad, hb = ho * s.stride - s.pad;
        for (int it = 0; it < nk; ++it, ++g) {
          const int st = (int)(g % C::STAGES);
          const int64_t use = g / C::STAGES;
          if (use >= 1) ptx::mbar_wait(&empty[st], (uint32_t)((use - 1) & 1));
          ptx::mbar_arrive_expect_tx(&full[st], iss2 ? CA_BYTES : C::STAGE);
#pragma unroll
          for (int h = 0; h < KB; ++h) {
            const int kbi = it * KB + h;
            const bool valid = kbi < a.nkb;
            const int kv = valid ? kbi : a.nkb - 1;  // tail of an odd range: re-load a valid A block, B is 0
            const int tap = kv / cb, c0 = (kv - tap * cb) * 64;
            const int r = a.r0 + tap / a.ns, q = a.s0 + tap % a.ns;
            ptx::tma_load_im2col_4d(&tmX, &full[st], sA + st * CA_BYTES + h * (CBM * CBK * 2), c0, wb, hb, nn,
                                    (uint16_t)q, (uint16_t)r);
            if (!iss2) {
              const int wcol = valid ? (r * s.kw + q) * s.C + c0 : a.K;  // column K: all out of bounds -> zeros
              ptx::tma_load_2d(&tmW, &full[st], sB + st * C::B_BYTES + h * C::B_ATOM, wcol, n0);
            }
          }
        }
      }
    }
  } else if (warp == 6) {
    // W issuer: the same tiles (a third reader of the tile ring) and the same stage sequence
    // (single-producer comparisons, a.dbg & 1: idle)
    int64_t g = 0;
    for (int j = 0; iss2; ++j) {
      const int slot = j & 3;
      ptx::mbar_wait(&tile_full[slot], (uint32_t)((j >> 2) & 1));
      const int u = s_tile[slot];
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&tile_empty[slot]);
      if (u < 0) break;
      const int n0 = (int)((int64_t)u % tiles_n) * BN;
      for (int it = 0; it < nk; ++it, ++g) {
        const int st = (int)(g % C::STAGES);
        const int64_t use = g / C::STAGES;
        if (use >= 1) ptx::mbar_wait(&empty[st], (uint32_t)((use - 1) & 1));
        if (lane == 0) {
          ptx::mbar_arrive_expect_tx(&full[st], C::B_BYTES);
#pragma unroll
          for (int h = 0; h < KB; ++h) {
            const int kbi = it * KB + h;
            const bool valid = kbi < a.nkb;
            const int kv = valid ? kbi : a.nkb - 1;
            const int tap = kv / cb, c0 = (kv - tap * cb) * 64;
            const int r = a.r0 + tap / a.ns, q = a.s0 + tap % a.ns;
            const int wcol = valid ? (r * s.kw + q) * s.C + c0 : a.K;
            ptx::tma_load_2d(&tmW, &full[st], sB + st * C::B_BYTES + h * C::B_ATOM, wcol, n0);
          }
        }
        __syncwarp();
      }
    }
  } else if (warp == 1) {
    // the whole warp walks the loop (uniform descriptors); elect.sync issues each UMMA
    constexpr uint32_t idesc = ptx::idesc_bf16(CBM, BN);
    const uint64_t da0 = ptx::desc_sw128(ptx::smem_u32(sA));
    const uint64_t db0 = ptx::desc_sw128(ptx::smem_u32(sB));
    int64_t g = 0;
    for (int j = 0;; ++j) {
      const int slot = j & 3;
      ptx::mbar_wait(&tile_full[slot], (uint32_t)((j >> 2) & 1));
      const int u = s_tile[slot];
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&tile_empty[slot]);
      if (u < 0) break;
      const int acc = j & 1;
      const int use_acc = j >> 1;
      if (use_acc >= 1) ptx::mbar_wait(&tmem_empty[acc], (use_acc - 1) & 1);
      ptx::tc_fence_after();
      const uint32_t d = tmem + acc * C::TMEM_COLS;
      for (int it = 0; it < nk; ++it, ++g) {
        const int st = (int)(g % C::STAGES);
        ptx::mbar_wait(&full[st], (uint32_t)((g / C::STAGES) & 1));
        ptx::tc_fence_after();
#pragma unroll
        for (int h = 0; h < KB; ++h) {
          // descriptor start address is bits [0, 14) in 16-byte units: offsets add directly
          const uint64_t da = da0 + (uint64_t)((st * CA_BYTES + h * (CBM * CBK * 2)) >> 4);
          const uint64_t db = db0 + (uint64_t)((st * C::B_BYTES + h * C::B_ATOM) >> 4);
#pragma unroll
          for (int k = 0; k < CBK / 16; ++k) ptx::umma_bf16_elect(d, da + 2 * k, db + 2 * k, idesc, (it | h | k) != 0);
        }
        ptx::umma_commit_elect(&empty[st]);
      }
      ptx::umma_commit_elect(&tmem_full[acc]);
    }
  } else {
    const int et = threadIdx.x - 64;
    const int qd = warp & 3;
    for (int j = 0;; ++j) {
      const int slot = j & 3;
      ptx::mbar_wait(&tile_full[slot], (uint32_t)((j >> 2) & 1));
      const int u = s_tile[slot];
      asm volatile("bar.sync 1, 128;" ::: "memory");  // every epilogue thread has read s_tile[slot]
      if (et == 0) ptx::mbar_arrive(&tile_empty[slot]);
      if (u < 0) break;
      const int acc = j & 1;
      const int64_t tile = u;
      const int n0 = (int)(tile % tiles_n) * BN;
      const int rt = qd * 32 + lane;  // row within the tile
      const int64_t row = (tile / tiles_n) * CBM + rt;
      for (int c = et; c < BN; c += 128) s_bias[c] = (n0 + c < s.Co) ? a.bias[n0 + c] : 0.0f;
      asm volatile("bar.sync 1, 128;" ::: "memory");
      ptx::mbar_wait(&tmem_full[acc], (j >> 1) & 1);
      ptx::tc_fence_after();
      const uint32_t tq = tmem + acc * C::TMEM_COLS + ((uint32_t)(qd * 32) << 16);
      __nv_bfloat16* out = a.y + row * s.Co;
      const __nv_bfloat16* res = a.res ? a.res + row * s.Co : nullptr;
      auto finish16 = [&](int c, float* v) {  // bias (+ residual) + activation + bf16 store of 16 columns
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
          bias_act<16>(v, s_bias + c * 16, a.act);
          store_row16_any(out + col0, v, s.Co - col0);
        }
      };
#pragma unroll 1
      for (int c = 0; c < BN / 16; ++c) {
        float v[16];
        ptx::tmem_ld16(tq + c * 16, v);
        finish16(c, v);
      }
      ptx::tc_fence_before();
      ptx::mbar_arrive(&tmem_empty[acc]);
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, 2 * C::TMEM_COLS);
  }
}

template <int BN, int OCC = 1, int KB = 2>
void launch_conv_tma(const CUtensorMap& tx, const CUtensorMap& tw, const ConvArgs& a, cudaStream_t st) {
  using C = ConvCfg<BN, OCC, KB>;
  auto kern = conv_tma_kernel<BN, OCC, KB>;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM));
    attr = true;
  }
  const int64_t M = (int64_t)a.s.N * a.s.Ho * a.s.Wo;
  const int64_t units = ((M + CBM - 1) / CBM) * ((a.s.Co + BN - 1) / BN);
  int dev = 0;
  cudaGetDevice(&dev);
  const int grid = (int)std::min<int64_t>(units, (int64_t)OCC * num_sms(dev));
  launch_pdl_if(pdl_on(true), kern, dim3(grid), dim3(conv_threads<OCC>()), C::SMEM, st, tx, tw, a);
}


PFN_cuTensorMapEncodeIm2col_v12000 get_encode_im2col() {
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

}  // namespace

ConvTaps conv_taps(const ConvShape& s) {
  // taps whose input row / column is in the padding for every output pixel contribute exact zeros
  ConvTaps t;
  t.r0 = std::max(0, s.pad - (s.Ho - 1) * s.stride);
  const int r1 = std::min(s.kh - 1, s.H - 1 + s.pad);
  t.s0 = std::max(0, s.pad - (s.Wo - 1) * s.stride);
  const int s1 = std::min(s.kw - 1, s.W - 1 + s.pad);
  t.nr = std::max(1, r1 - t.r0 + 1);
  t.ns = std::max(1, s1 - t.s0 + 1);
  return t;
}

ConvPlan conv_tc_plan(const ConvShape& s, int sms) {
  // tile width: measured at every c4 / c5 ResNet shape (tools/plan_sweep.sh, DESIGN.md "Conv design
  // notes"), 128-wide tiles beat 64 (narrow tiles pay the per-k-block cost twice per FLOP) and 256
  // (half the CTAs on these grids); 64 only for 64-channel layers
  const ConvTaps t = conv_taps(s);
  (void)sms;
  return ConvPlan{s.Co <= 64 ? 64 : 128, 1, t.nr * t.ns * (s.C / 64)};
}

int conv_tc_pick_bn(const ConvShape& s, int sms) { return conv_tc_plan(s, sms).bn; }

bool conv_tma_ok(const ConvShape& s) { return s.C % 64 == 0 && s.kh <= 16 && s.kw <= 16; }

CUtensorMap make_tmap_im2col(const void* x, const ConvShape& s) {
  CUtensorMap m;
  cuuint64_t dims[4] = {(cuuint64_t)s.C, (cuuint64_t)s.W, (cuuint64_t)s.H, (cuuint64_t)s.N};
  cuuint64_t strides[3] = {(cuuint64_t)s.C * 2, (cuuint64_t)s.W * s.C * 2, (cuuint64_t)s.H * s.W * s.C * 2};
  int lower[2] = {-s.pad, -s.pad};                                // (W, H)
  int upper[2] = {s.pad - (s.kw - 1), s.pad - (s.kh - 1)};
  cuuint32_t estr[4] = {1, (cuuint32_t)s.stride, (cuuint32_t)s.stride, 1};
  CUresult r = get_encode_im2col()(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(x), dims, strides, lower,
                                   upper, 64, CBM, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) fail(DUET_ECUDA, "cuTensorMapEncodeIm2col failed (" + std::to_string((int)r) + ")");
  // Same driver workaround CUTLASS applies (copy_traits_sm90_im2col.hpp): for tensors < 128 KiB on
  // drivers <= 13.1 clear bit 21 of descriptor word 1.
  int drv = 0;
  cudaDriverGetVersion(&drv);
  if (drv <= 13010 && (int64_t)s.N * s.H * s.W * s.C * 2 < 131072) reinterpret_cast<uint64_t*>(&m)[1] &= ~(1ull << 21);
  return m;
}

void conv_tc(const CUtensorMap& tw, const void* x, const float* bias, const void* residual, void* y,
             const ConvShape& s, int K, int act, const ConvPlan& p, unsigned* ctr, cudaStream_t st) {
  const ConvTaps t = conv_taps(s);
  static const int iss_env = getenv("DUET_CONV_ISS") ? atoi(getenv("DUET_CONV_ISS")) : 2;
  ConvArgs a{(const __nv_bfloat16*)x, bias, (const __nv_bfloat16*)residual, (__nv_bfloat16*)y, s, K, act,
             p.nkb, t.r0, t.s0, t.ns, ctr, iss_env == 1 ? 1 : 0};
  const int bn = p.bn;
  if (conv_tma_ok(s) && ((uintptr_t)x % 16) == 0) {
    CUtensorMap tx = make_tmap_im2col(x, s);
    switch (bn) {
      case 64: {
        // several CTAs per SM for the 64-channel layers: their tiles are bound by per-tile TMA round
        // trips, and independent CTAs (each its own ring, MMA warp and epilogue) overlap them.
        // Measured (conv_one, CUDA graphs, same box; profiles/r2_conv_occ.log): c5 layer 1 (4096 x
        // 8x8x64) 1 CTA 70.6, 2 CTAs 37.6, 3 CTAs with one-k-block stages 32.8, 4 CTAs 33.5 us;
        // c4 layer 1 (64 x 56x56x64) 31.5 / 26.9 / 28.2 us (the SMEM-halo kernel 30.0).
        // DUET_CONV_OCC: 1, 2 (two-k-block stages), 4 = that many CTAs; default 3
        static const int occ = getenv("DUET_CONV_OCC") ? atoi(getenv("DUET_CONV_OCC")) : 3;
        if (occ == 1) return launch_conv_tma<64>(tx, tw, a, st);
        if (occ == 2) return launch_conv_tma<64, 2>(tx, tw, a, st);
        if (occ == 4) return launch_conv_tma<64, 4, 1>(tx, tw, a, st);
        return launch_conv_tma<64, 3, 1>(tx, tw, a, st);
      }
      // (two CTAs per SM with one-k-block stages for 128-wide tiles measured -9% .. +18% across
      // the c4 / c5 shapes and c4 p50 unchanged: not used, profiles/r2_conv.md)
      case 128: {
        // two CTAs per SM (one-k-block stages) once the tiles outnumber the SMs (with fewer, the
        // second CTA of an SM only halves the first's share): c5 layer 3 (4096 x 2x2x256) 26.1 ->
        // 21.8 us, layer 2 27.5 -> 24.7, c4 layer 3 25.7 -> 21.9, layer 2 22.4 -> 21.3; c4 layer 4
        // (100 tiles) 25.2 -> 33.0 with two, so it keeps one (profiles/r2_conv_occ128.log).
        // DUET_CONV_OCC128: 1 / 2 force one / two CTAs per SM
        static const int occ128 = getenv("DUET_CONV_OCC128") ? atoi(getenv("DUET_CONV_OCC128")) : 0;
        const int64_t M = (int64_t)s.N * s.Ho * s.Wo;
        const int64_t tiles = ((M + CBM - 1) / CBM) * ((s.Co + 127) / 128);
        int dev = 0;
        cudaGetDevice(&dev);
        const bool two = occ128 == 2 || (occ128 == 0 && tiles > num_sms(dev));
        if (two) return launch_conv_tma<128, 2, 1>(tx, tw, a, st);
        return launch_conv_tma<128>(tx, tw, a, st);
      }
      case 256: return launch_conv_tma<256>(tx, tw, a, st);
    }
  }
  fail(DUET_EUNSUPPORTED, "conv_tc: needs C % 64 == 0 (16-B aligned input) and bn in {64, 128, 256}");
}

}  // namespace duet
