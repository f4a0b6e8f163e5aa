// Halo implicit-GEMM 3x3 / stride-1 / pad-1 convolution on tcgen05 (DESIGN.md
// "Conv design notes", round 2).
//
// The im2col-TMA kernel (conv_tc.cu) loads, per 64-channel filter tap, 128 output pixels' input rows:
// every input pixel crosses L2 -> SMEM nine times, as 128-byte segments, and ResNet's 64-128-channel
// layers were bound by that segment stream (c4 layer 1: 0.18 of the tensor peak, tensor pipe ~4%).
// Here the input tile is loaded ONCE per 64-channel block, with its one-pixel halo, by a tiled TMA
// whose out-of-image coordinates are zero-filled -- i.e. the zero padding is materialised in shared
// memory -- and the nine taps are read from it:
//
//   padded input rows  p = (img * Hs + yy) * Wp + xx      (Wp = W + 2, Hs = rows per image block)
//   output rows        m = (img * Hs + y)  * Wp + x       (y < hb, x < W valid; the rest garbage)
//   tap (r, s) reads   p = m + r * Wp + s                  -> a CONTIGUOUS 128-row window
//
// so each tap's A operand is the same SMEM buffer with its start moved by (r Wp + s) rows of 128 B
// (UMMA descriptor start address; the swizzle phase follows the absolute address, see desc_sw128_at).  Garbage rows
// (x >= W, the last two rows of an image block) are computed and discarded by the epilogue.  A work
// unit is a band of hb output rows of one image (hb Wp <= 128) or, for small maps, ni whole images.
// The BN-folded weights are either resident in SMEM for the whole kernel (C = 64, BN = 64: 72 KB)
// or streamed per (tap, channel block) through a ring.  Epilogue as conv_tc.cu: bias + residual +
// ReLU, bf16 NHWC stores of the valid rows.
#include <cudaTypedefs.h>

#include "../common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace duet {

namespace {

constexpr int HBM_ROWS = 128;  // UMMA M
constexpr int kHaloSmem = 220 * 1024;

struct HaloArgs {
  const __nv_bfloat16* bias_dummy;
  const float* bias;
  const __nv_bfloat16* res;
  __nv_bfloat16* y;
  ConvShape s;
  int act;
  int Wp;          // W + 2
  int Hs;          // padded rows per image block in SMEM (hb + 2)
  int hb;          // output rows per unit per image
  int ni;          // images per unit
  int bands;       // units per image (ni == 1), else 1
  int a_bytes;     // one A stage (>= box bytes, >= (128 + 2 Wp + 2) rows), multiple of 1024
  int box_bytes;   // bytes the halo TMA delivers (zero-filled halo included)
  int a_stages, b_stages;
  int bres;        // weights resident in SMEM
  unsigned* ctr;   // [2] dynamic unit counter + exit count (null: static units block + j grid)
};

// SWIZZLE_128B K-major descriptor whose start sits at any 128-B row of a 1024-B aligned buffer the
// TMA filled: the UMMA unit applies the swizzle XOR from the ABSOLUTE address bits (like the TMA
// that wrote it), so the start address alone moves the window and the matrix base offset stays 0.
// (Measured on the B200: base offset = (addr >> 7) & 7 -- the reading of "not aligned to the
// pattern boundary" -- gives garbage; 0 is exact.)
__device__ __forceinline__ uint64_t desc_sw128_at(uint32_t saddr) { return ptx::desc_sw128(saddr); }

template <int BN>
__global__ void __launch_bounds__(192, 1) conv_halo_kernel(const __grid_constant__ CUtensorMap tmX,
                                                           const __grid_constant__ CUtensorMap tmW, const HaloArgs a) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  constexpr int B_BLOCK = BN * 128;  // one 64-wide k-block of BN weight rows
  const ConvShape& s = a.s;
  const int cb = s.C / 64;
  const int nkw = 9 * cb;
  uint8_t* sA = smem;
  uint8_t* sB = smem + a.a_stages * a.a_bytes;
  const int b_slots = a.bres ? nkw : a.b_stages;
  uint64_t* a_full = reinterpret_cast<uint64_t*>(sB + b_slots * B_BLOCK);
  uint64_t* a_empty = a_full + 4;
  uint64_t* b_full = a_empty + 4;
  uint64_t* b_empty = b_full + 8;
  uint64_t* tmem_full = b_empty + 8;
  uint64_t* tmem_empty = tmem_full + 2;
  uint64_t* w_full = tmem_empty + 2;
  uint64_t* u_full = w_full + 1;   // [4] unit ring (dynamic scheduling, as conv_tc.cu)
  uint64_t* u_empty = u_full + 4;  // [4]
  int* s_unit = reinterpret_cast<int*>(u_empty + 4);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(s_unit + 4);
  float* s_bias = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(a_full) + 512);

  const int warp = ptx::warp_id();
  const int lane = threadIdx.x & 31;
  const int tiles_n = (s.Co + BN - 1) / BN;
  const int64_t groups = a.ni == 1 ? (int64_t)s.N * a.bands : ((int64_t)s.N + a.ni - 1) / a.ni;
  const int64_t n_units = groups * tiles_n;
  constexpr int TMEM_COLS = BN <= 64 ? 64 : BN <= 128 ? 128 : 256;
  auto unit_geo = [&](int64_t u, int& n0, int& y0, int& nt) {
    nt = (int)(u % tiles_n);
    const int64_t gi = u / tiles_n;
    if (a.ni == 1) {
      n0 = (int)(gi / a.bands);
      y0 = (int)(gi % a.bands) * a.hb;
    } else {
      n0 = (int)(gi * a.ni);
      y0 = 0;
    }
  };

  if (threadIdx.x == 0) {
    ptx::tma_prefetch(&tmX);
    ptx::tma_prefetch(&tmW);
    for (int i = 0; i < a.a_stages; ++i) {
      ptx::mbar_init(&a_full[i], 1);
      ptx::mbar_init(&a_empty[i], 1);
    }
    for (int i = 0; i < a.b_stages; ++i) {
      ptx::mbar_init(&b_full[i], 1);
      ptx::mbar_init(&b_empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(&tmem_full[i], 1);
      ptx::mbar_init(&tmem_empty[i], 128);
    }
    ptx::mbar_init(w_full, 1);
    for (int i = 0; i < 4; ++i) {
      ptx::mbar_init(&u_full[i], 1);
      ptx::mbar_init(&u_empty[i], 2);
    }
    ptx::fence_mbar_init();
  }
  ptx::pdl_wait();  // before tensor memory is taken
  if (warp == 1) {
    ptx::tmem_alloc(tmem_slot, 2 * TMEM_COLS);
    ptx::tmem_relinquish();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  ptx::pdl_trigger();

  if (warp == 0) {
    if (lane == 0) {
      if (a.bres) {  // every weight block of the (single) n tile, once
        ptx::mbar_arrive_expect_tx(w_full, (uint32_t)(nkw * B_BLOCK));
        for (int j = 0; j < nkw; ++j) ptx::tma_load_2d(&tmW, w_full, sB + j * B_BLOCK, j * 64, 0);
      }
      int64_t ga = 0, gb = 0;
      for (int j = 0;; ++j) {
        int64_t u = a.ctr ? (int64_t)atomicAdd(a.ctr, 1u) : (int64_t)blockIdx.x + (int64_t)j * gridDim.x;
        const int slot = j & 3;
        if (j >= 4) ptx::mbar_wait(&u_empty[slot], (uint32_t)(((j >> 2) - 1) & 1));
        s_unit[slot] = u < n_units ? (int)u : -1;
        ptx::mbar_arrive(&u_full[slot]);
        if (u >= n_units) {
          if (a.ctr && atomicAdd(a.ctr + 1, 1u) == gridDim.x - 1) {  // last CTA done fetching: reset
            a.ctr[0] = 0;
            a.ctr[1] = 0;
          }
          break;
        }
        int n0, y0, nt;
        unit_geo(u, n0, y0, nt);
        for (int c = 0; c < cb; ++c, ++ga) {
          const int st = (int)(ga % a.a_stages);
          const int64_t use = ga / a.a_stages;
          if (use >= 1) ptx::mbar_wait(&a_empty[st], (uint32_t)((use - 1) & 1));
          ptx::mbar_arrive_expect_tx(&a_full[st], (uint32_t)a.box_bytes);
          // box (64 ch, Wp, Hs, ni) at (c*64, -1, y0-1, n0): the halo outside the image is zero-filled
          asm volatile(
              "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, "
              "%6}], [%2];" ::"r"(ptx::smem_u32(sA + (size_t)st * a.a_bytes)),
              "l"((uint64_t)&tmX), "r"(ptx::smem_u32(&a_full[st])), "r"(c * 64), "r"(-1), "r"(y0 - 1), "r"(n0)
              : "memory");
          if (!a.bres) {
            for (int tap = 0; tap < 9; ++tap, ++gb) {
              const int bs = (int)(gb % a.b_stages);
              const int64_t ub = gb / a.b_stages;
              if (ub >= 1) ptx::mbar_wait(&b_empty[bs], (uint32_t)((ub - 1) & 1));
              ptx::mbar_arrive_expect_tx(&b_full[bs], (uint32_t)B_BLOCK);
              ptx::tma_load_2d(&tmW, &b_full[bs], sB + bs * B_BLOCK, (tap * cb + c) * 64, nt * BN);
            }
          }
        }
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t idesc = ptx::idesc_bf16(HBM_ROWS, BN);
    const uint32_t a_base = ptx::smem_u32(sA);
    const uint64_t db0 = ptx::desc_sw128(ptx::smem_u32(sB));
    if (a.bres) ptx::mbar_wait(w_full, 0);
    int64_t ga = 0, gb = 0;
    for (int j = 0;; ++j) {
      ptx::mbar_wait(&u_full[j & 3], (uint32_t)((j >> 2) & 1));
      const int u = s_unit[j & 3];
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&u_empty[j & 3]);
      if (u < 0) break;
      const int acc = j & 1;
      if ((j >> 1) >= 1) ptx::mbar_wait(&tmem_empty[acc], ((j >> 1) - 1) & 1);
      ptx::tc_fence_after();
      const uint32_t d = tmem + acc * TMEM_COLS;
      for (int c = 0; c < cb; ++c, ++ga) {
        const int st = (int)(ga % a.a_stages);
        ptx::mbar_wait(&a_full[st], (uint32_t)((ga / a.a_stages) & 1));
        ptx::tc_fence_after();
        const uint32_t abuf = a_base + (uint32_t)(st * a.a_bytes);
        for (int tap = 0; tap < 9; ++tap) {
          const int r = tap / 3, q = tap - r * 3;
          int bs = 0;
          if (!a.bres) {
            bs = (int)(gb % a.b_stages);
            ptx::mbar_wait(&b_full[bs], (uint32_t)((gb / a.b_stages) & 1));
            ptx::tc_fence_after();
          }
          const uint64_t da = desc_sw128_at(abuf + (uint32_t)((r * a.Wp + q) * 128));
          const uint64_t db = db0 + (uint64_t)(((a.bres ? tap * cb + c : bs) * B_BLOCK) >> 4);
#pragma unroll
          for (int k = 0; k < 4; ++k) ptx::umma_bf16_elect(d, da + 2 * k, db + 2 * k, idesc, (c | tap | k) != 0);
          if (!a.bres) {
            ptx::umma_commit_elect(&b_empty[bs]);
            ++gb;
          }
        }
        ptx::umma_commit_elect(&a_empty[st]);
      }
      ptx::umma_commit_elect(&tmem_full[acc]);
    }
  } else {
    const int et = threadIdx.x - 64;
    const int qd = warp & 3;
    const int m = qd * 32 + lane;  // accumulator row = output row within the unit
    const int img_rows = a.Hs * a.Wp;
    const int img = m / img_rows;
    const int yy = (m - img * img_rows) / a.Wp;
    const int xx = m - img * img_rows - yy * a.Wp;
    for (int j = 0;; ++j) {
      ptx::mbar_wait(&u_full[j & 3], (uint32_t)((j >> 2) & 1));
      const int u = s_unit[j & 3];
      asm volatile("bar.sync 1, 128;" ::: "memory");  // every epilogue thread has read the unit
      if (et == 0) ptx::mbar_arrive(&u_empty[j & 3]);
      if (u < 0) break;
      const int acc = j & 1;
      int n0, y0, nt;
      unit_geo(u, n0, y0, nt);
      const int nb = nt * BN;
      for (int c = et; c < BN; c += 128) s_bias[c] = (nb + c < s.Co) ? a.bias[nb + c] : 0.0f;
      asm volatile("bar.sync 1, 128;" ::: "memory");
      ptx::mbar_wait(&tmem_full[acc], (j >> 1) & 1);
      ptx::tc_fence_after();
      const bool valid = img < a.ni && n0 + img < s.N && yy < a.hb && y0 + yy < s.H && xx < s.W;
      const int64_t orow = valid ? ((int64_t)(n0 + img) * s.H + y0 + yy) * s.W + xx : 0;
      const uint32_t tq = tmem + acc * TMEM_COLS + ((uint32_t)(qd * 32) << 16);
      __nv_bfloat16* out = a.y + orow * s.Co;
      const __nv_bfloat16* res = a.res ? a.res + orow * s.Co : nullptr;
#pragma unroll 1
      for (int c = 0; c < BN / 16; ++c) {
        float v[16];
        ptx::tmem_ld16(tq + c * 16, v);
        const int col0 = nb + c * 16;
        if (valid && col0 < s.Co) {
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
      }
      ptx::tc_fence_before();
      ptx::mbar_arrive(&tmem_empty[acc]);
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, 2 * TMEM_COLS);
  }
}

}  // namespace

HaloPlan conv_halo_plan(const ConvShape& s, int sms, bool force) {
  HaloPlan p;
  if (s.stride != 1 || s.kh != 3 || s.kw != 3 || s.pad != 1 || s.C % 64 || s.Co % 16 || s.C > 512) return p;
  const int Wp = s.W + 2;
  if (Wp > 126) return p;
  int hb, ni, Hs;
  if (s.H * Wp <= HBM_ROWS) {  // whole images per unit
    hb = s.H;
    Hs = s.H + 2;
    ni = (HBM_ROWS - s.H * Wp) / (Hs * Wp) + 1;
    if (ni > s.N) ni = s.N;
  } else {
    hb = HBM_ROWS / Wp;
    Hs = hb + 2;
    ni = 1;
  }
  if (hb < 1 || Hs > 256 || ni > 256) return p;
  const int bands = ni == 1 ? (s.H + hb - 1) / hb : 1;
  const int64_t groups = ni == 1 ? (int64_t)s.N * bands : ((int64_t)s.N + ni - 1) / ni;
  const double valid = (double)s.N * s.H * s.W / ((double)groups * HBM_ROWS);
  if (valid < 0.45 && !force) return p;
  int bn = s.Co <= 64 ? 64 : s.Co <= 128 ? 128 : 256;
  if (bn == 256 && groups * 2 >= sms) bn = 128;  // narrower tiles when there is enough work
  const int box_rows = ni * Hs * Wp;
  const int need_rows = std::max(box_rows, HBM_ROWS + 2 * Wp + 2 + 8);
  const int a_bytes = ((need_rows * 128) + 1023) / 1024 * 1024;
  const int b_block = bn * 128;
  const int nkw = 9 * (s.C / 64);
  const int bres = (s.Co <= bn && nkw * b_block <= 96 * 1024) ? 1 : 0;
  const int fixed = 2048 + bn * 4;
  int a_st = 2, b_st = 0;
  if (bres) {
    a_st = std::min(4, (kHaloSmem - fixed - nkw * b_block) / a_bytes);
  } else {
    a_st = std::min(3, std::max(2, (kHaloSmem - fixed - 4 * b_block) / a_bytes));
    b_st = std::min(8, (kHaloSmem - fixed - a_st * a_bytes) / b_block);
  }
  if (a_st < 2 || (!bres && b_st < 3)) return p;
  p.ok = true;
  // measured (ncu, profiles/r2_conv.md): the halo kernel wins where the weights stay resident and
  // the band holds >= 2 image rows of >= 16 pixels (c4 layer 1: 40 -> 33 us); with streamed
  // weights (128-256 channels) or 8 x 8 maps (50% valid rows) the im2col-TMA kernel is faster
  if ((!bres || s.W < 16) && !force) {
    p.ok = false;
    return p;
  }
  p.bn = bn;
  p.hb = hb;
  p.ni = ni;
  p.Hs = Hs;
  p.bands = bands;
  p.a_bytes = a_bytes;
  p.box_bytes = box_rows * 128;
  p.a_stages = a_st;
  p.b_stages = bres ? 1 : b_st;
  p.bres = bres;
  p.smem = 1024 + a_st * a_bytes + (bres ? nkw : b_st) * b_block + fixed;
  p.units = groups * ((s.Co + bn - 1) / bn);
  return p;
}

void conv_halo(const CUtensorMap& tw, const void* x, const float* bias, const void* residual, void* y, const ConvShape& s,
               int act, const HaloPlan& p, unsigned* ctr, cudaStream_t st) {
  if (!p.ok) fail(DUET_EINVAL, "conv_halo: shape not eligible");
  if (((uintptr_t)x & 15) || ((uintptr_t)y & 15)) fail(DUET_EUNSUPPORTED, "conv_halo: 16-B aligned tensors");
  CUtensorMap tx;
  cuuint64_t dims[4] = {(cuuint64_t)s.C, (cuuint64_t)s.W, (cuuint64_t)s.H, (cuuint64_t)s.N};
  cuuint64_t strides[3] = {(cuuint64_t)s.C * 2, (cuuint64_t)s.W * s.C * 2, (cuuint64_t)s.H * s.W * s.C * 2};
  cuuint32_t box[4] = {64, (cuuint32_t)(s.W + 2), (cuuint32_t)p.Hs, (cuuint32_t)p.ni};
  cuuint32_t estr[4] = {1, 1, 1, 1};
  CUresult r = tmap_encode_tiled()(&tx, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(x), dims, strides, box,
                                   estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) fail(DUET_ECUDA, "conv_halo: cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ")");
  HaloArgs a{nullptr, bias, (const __nv_bfloat16*)residual, (__nv_bfloat16*)y, s, act, s.W + 2, p.Hs, p.hb, p.ni,
             p.bands, p.a_bytes, p.box_bytes, p.a_stages, p.b_stages, p.bres, ctr};
  int dev = 0;
  cudaGetDevice(&dev);
  const int grid = (int)std::min<int64_t>(p.units, num_sms(dev));
  auto go = [&](auto kern) {
    static int attr = 0;  // per instantiation: the largest dynamic smem granted so far
    if (p.smem > attr) {
      CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem));
      attr = p.smem;
    }
    launch_pdl_if(pdl_on(true), kern, dim3(grid), dim3(192), (size_t)p.smem, st, tx, tw, a);
  };
  switch (p.bn) {
    case 64: go(conv_halo_kernel<64>); break;
    case 128: go(conv_halo_kernel<128>); break;
    case 256: go(conv_halo_kernel<256>); break;
    default: fail(DUET_EINVAL, "conv_halo: bn");
  }
}

}  // namespace duet
