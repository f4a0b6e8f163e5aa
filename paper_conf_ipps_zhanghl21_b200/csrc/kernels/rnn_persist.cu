// Persistent fused LSTM / GRU recurrence for latency-bound batches.
//
// One launch runs all S time steps.  CTA (n, m) owns gate-block tile n (U = BN/4 hidden units,
// all four gate blocks, the same packed weights as the per-step kernel in gemm_tc.cu) for batch
// rows [128 m, +128).  Per step t:
//
//   acc[t&1]  = x_t W_x^T              (kx k-blocks; independent of h, so they are loaded and
//                                       multiplied while step t-1's epilogue and barrier run)
//   acc[t&1] += h_{t-1} W_h^T          (kh k-blocks, loaded by TMA after the grid barrier)
//   epilogue: gates -> c_t (LSTM, fp32 in registers for the whole sequence), h_t -> bf16 global
//   grid barrier: every CTA's slice of h_t is written (one release-add per epilogue warp per step)
//
// Versus one kernel per step this removes the launch / prologue / TMEM allocation of every step
// and the x-projection from the critical path; the cell state never leaves the SM.  The TMEM
// accumulator is double-buffered (2 x BN columns) so step t+1's x part overlaps step t's epilogue.
// Co-residency of the grid (required by the barrier) is guaranteed by a cooperative launch; the
// runtime uses this kernel only when the grid fits in half of the SMs (two recurrent branches on
// two stream slots must co-reside).
//
// Warp roles: warp 0 TMA producer, warp 1 TMEM allocator + MMA issuer (warp-convergent, elect.sync),
// warps 2..9 epilogue (warp w reads TMEM lane quarter w % 4; the two warps of a quarter split the
// units of the tile).
#include "../common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace duet {

// per-CTA, per-step %globaltimer stamps when RnnPersistArgs::dbg & 1 (tools/rnn_trace.py):
// [cta][t][0] h_{t-1} barrier passed (producer), [1] first x stage landed (MMA warp),
// [2] accumulator ready (epilogue), [3] h_t stored + released (epilogue), [4] first h stage landed
// (MMA warp), [5] last UMMA of the step issued
__device__ unsigned long long g_rp_trace[128 * 64 * 16];

namespace {

__device__ __forceinline__ unsigned long long rp_gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

constexpr int RBM = 128;
constexpr int RBK = 64;
constexpr int R_A_BYTES = RBM * RBK * 2;
constexpr int kREpiWarps = 8;
constexpr int kRThreads = 64 + 32 * kREpiWarps + 32 + 32;  // + W producer, second A issuer
constexpr int kWWarp = 2 + kREpiWarps;
// Second TMA issuer (round 2, a.issue2): one thread's bulk / tensor copies into an SM complete in
// issue order at ~16 KB per 0.37 us (~44 GB/s) whatever their size, so the x / h stream gets a
// second issuing warp that takes the odd ring stages (measured on the c3 tower with the resident-W
// warp issuing every other h block: 381 -> 336 us).  (A thirteenth
// warp would round the register budget down to 128 per thread: spills.)
constexpr int kA2Warp = kWWarp + 1;

template <int BN>
struct RCfg {
  static constexpr int U = BN / 4;   // hidden units per tile
  static constexpr int UH = U / 2;   // units per epilogue thread
  static constexpr int B_BYTES = BN * RBK * 2;
  static constexpr int TMEM_COLS = 2 * BN <= 128 ? 128 : 2 * BN <= 256 ? 256 : 512;
  static constexpr int EXTRA = 1024 + 512 + BN * 4;  // alignment slack + barriers + bias
};
// Shared-memory plan: [A ring: stages x 16 KB][W: resident (kx + kh blocks) or a ring of `stages`
// blocks][barriers][bias].  W is resident when it fits next to a ring of >= 6 A stages.
constexpr int kRSmemBudget = 227 * 1024;
inline int rp_plan(int bn, int nkw, bool* wres, int min_res_stages = 6) {
  const int bb = bn * RBK * 2, extra = 1024 + 512 + bn * 4;
  const int res_stages = (kRSmemBudget - extra - nkw * bb) / R_A_BYTES;
  if (res_stages >= min_res_stages) {
    *wres = true;
    return res_stages > 10 ? 10 : res_stages;
  }
  *wres = false;
  const int st = (192 * 1024) / (R_A_BYTES + bb);
  return st > 10 ? 10 : st;
}

// (measured: a relaxed polling loop + one fence.acq_rel.gpu passes the barrier ~0.3 us later than
// polling with ld.acquire)
__device__ __forceinline__ unsigned ld_relaxed_gpu(const unsigned* p) {
  unsigned v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned ld_acquire_gpu(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void red_release_gpu_add(unsigned* p, unsigned v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

__device__ __forceinline__ float tanh_approx(float x) {
  float y;
  asm("tanh.approx.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
// bf16 path only (tolerance 2e-2): tanh.approx.f32 has ~2^-11 relative error,
// below the bf16 rounding of h_t itself
// sigma(x) = 0.5 tanh(x / 2) + 0.5: one MUFU op instead of ex2 + rcp (the epilogue is MUFU-bound:
// 2048 cells x 5 transcendental per CTA per step)
__device__ __forceinline__ float rsig(float x) { return fmaf(0.5f, tanh_approx(0.5f * x), 0.5f); }
__device__ __forceinline__ float rtanh(float x) { return tanh_approx(x); }

// mbarrier wait with the hardware suspend of try_wait: ten warps wait at different times here, and
// a spinning test_wait loop steals issue slots from the epilogue warps on the same SM sub-partition
__device__ __forceinline__ void wait_sleep(uint64_t* bar, uint32_t parity) {
  const uint32_t addr = ptx::smem_u32(bar);
  while (!ptx::mbar_try_wait(addr, parity)) {
  }
}

// one LSTM / GRU cell from its four gate pre-activations; `st` = c (LSTM) or h_{t-1} (GRU), updated
template <int KIND>
__device__ __forceinline__ float cell(float a0, float a1, float a2, float a3, float& st) {
  if constexpr (KIND == EPI_LSTM) {
    const float ig = rsig(a0), fg = rsig(a1), gg = rtanh(a2), og = rsig(a3);
    st = fg * st + ig * gg;
    return og * rtanh(st);
  } else {
    const float r = rsig(a0), z = rsig(a1);
    const float n = rtanh(a2 + r * a3);  // (W_in x + b_in) + r * (W_hn h + b_hn)
    const float h = (1.0f - z) * n + z * st;
    st = h;
    return h;
  }
}
// h_t buffers are K-blocked and pre-swizzled: [kh][Bp][64] with the 16-byte chunk c of row r at
// position c ^ (r & 7), i.e. exactly the SWIZZLE_128B K-major layout UMMA reads.  A (k-block, row
// tile) of h is then one contiguous 16 KB range, fetched with a single bulk copy instead of a
// 128-row tensor-map load.  Element index of the 8-unit group starting at `unit` (unit % 8 == 0):
__device__ __forceinline__ size_t hs_index(int row, int unit, int Bp) {
  return ((size_t)(unit >> 6) * Bp + row) * 64 + (size_t)((((unit & 63) >> 3) ^ (row & 7)) << 3);
}
__device__ __forceinline__ void store_bf16x8(__nv_bfloat16* dst, const float* h) {
  uint32_t w[4];
#pragma unroll
  for (int p = 0; p < 4; ++p) {
    __nv_bfloat162 b2 = __floats2bfloat162_rn(h[2 * p], h[2 * p + 1]);
    w[p] = *reinterpret_cast<uint32_t*>(&b2);
  }
  *reinterpret_cast<uint4*>(dst) = make_uint4(w[0], w[1], w[2], w[3]);
}

// the four gate blocks (N columns each, U apart) behind a single wait::ld
template <int N>
__device__ __forceinline__ void tmem_ld_gates(uint32_t taddr, int U, float (*v)[N]) {
  if constexpr (N == 8) {
    ptx::tmem_ld8x4(taddr, taddr + U, taddr + 2 * U, taddr + 3 * U, v);
  } else {
    uint32_t r[4][16];
#pragma unroll
    for (int g = 0; g < 4; ++g) ptx::tmem_ld16_nowait(taddr + g * U, r[g]);
#pragma unroll
    for (int g = 0; g < 4; ++g) ptx::tmem_wait_ld16(r[g]);  // the first waits, the rest pin the registers
#pragma unroll
    for (int g = 0; g < 4; ++g)
#pragma unroll
      for (int i = 0; i < 16; ++i) v[g][i] = __uint_as_float(r[g][i]);
  }
}
template <int N>
__device__ __forceinline__ void tmem_ld_n(uint32_t taddr, float* v) {
  if constexpr (N == 16) ptx::tmem_ld16(taddr, v);
  else ptx::tmem_ld8(taddr, v);
}

template <int BN, int KIND, bool WRES, bool MULTI>
__global__ void __launch_bounds__(kRThreads, 1)
    rnn_persist_kernel(const __grid_constant__ CUtensorMap tmX, const __grid_constant__ CUtensorMap tmH0,
                       const __grid_constant__ CUtensorMap tmH1, const __grid_constant__ CUtensorMap tmW,
                       const RnnPersistArgs a) {
  using C = RCfg<BN>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int STAGES = a.stages;
  const int nkw = a.kx + a.kh;  // packed weight k-blocks
  uint8_t* sA = smem;
  uint8_t* sB = smem + STAGES * R_A_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(sB + (WRES ? nkw : STAGES) * C::B_BYTES);
  uint64_t* empty = full + 10;
  uint64_t* tfull = empty + 10;
  uint64_t* tempty = tfull + 2;
  uint64_t* w_full = tempty + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(w_full + 1);
  float* s_bias = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(full) + 512);

  const int warp = ptx::warp_id();
  const int lane = threadIdx.x & 31;
  const int S = a.S, kx = a.kx, kh = a.kh;
  // static tile assignment: tile = blockIdx.x + i * gridDim.x (n-tile fastest); one tile per CTA
  // unless MULTI
  const int n_tiles = a.tiles_n * a.tiles_m;
  const int my_tiles = MULTI ? (n_tiles - 1 - (int)blockIdx.x) / (int)gridDim.x + 1 : 1;
  auto tile_n0 = [&](int i) { return ((int)(blockIdx.x + i * gridDim.x) % a.tiles_n) * BN; };
  auto tile_m0 = [&](int i) { return ((int)(blockIdx.x + i * gridDim.x) / a.tiles_n) * RBM; };
  const int cta = blockIdx.x;
  // packed k-block of the j-th load of a step: x blocks in order, then the h blocks rotated by
  // a.hrot * CTA (all CTAs reading the same 16 KB h block at once queue on the same L2 lines)
  const int hrot = kh > 0 ? (a.hrot * cta) % kh : 0;
  auto kblk = [&](int j) { return j < kx ? j : kx + (j - kx + hrot) % kh; };
  unsigned long long* trace = (a.dbg & 1) && !MULTI && cta < 128 ? g_rp_trace + (size_t)cta * 64 * 16 : nullptr;
  // several tiles per CTA: stamps per work unit u = t * my_tiles + i < 64 (tools/rnn_trace_multi.py):
  // 0 barrier observed (i = 0), 7 first A load issued, 11 first W load issued, 1 first stage landed,
  // 4 first h stage landed, 5 last UMMA issued, 2 accumulator ready, 6 TMEM read, 3 released
  unsigned long long* mtr = (a.dbg & 1) && MULTI && cta < 128 ? g_rp_trace + (size_t)cta * 64 * 16 : nullptr;

  if (threadIdx.x == 0) {
    ptx::tma_prefetch(&tmX);
    ptx::tma_prefetch(&tmH0);
    ptx::tma_prefetch(&tmH1);
    ptx::tma_prefetch(&tmW);
    for (int s = 0; s < STAGES; ++s) {
      ptx::mbar_init(&full[s], WRES ? 1 : 2);  // A producer (+ W producer), each with its tx bytes
      ptx::mbar_init(&empty[s], 1);
    }
    ptx::mbar_init(w_full, 1);
    for (int b = 0; b < 2; ++b) {
      ptx::mbar_init(&tfull[b], 1);
      ptx::mbar_init(&tempty[b], kREpiWarps);
    }
    ptx::fence_mbar_init();
  }
  if (warp == 1) {
    ptx::tmem_alloc(tmem_slot, C::TMEM_COLS);
    ptx::tmem_relinquish();
  }
  if (!MULTI)
    for (int c = (int)threadIdx.x - 64; c >= 0 && c < BN; c += 32 * kREpiWarps) s_bias[c] = a.bias[tile_n0(0) + c];
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0 || warp == kA2Warp) {
    // ---------------- A producer: x_t blocks, [grid barrier], h_{t-1} blocks per (step, tile) ------
    // (a.issue2: warp 0 issues the even ring stages, kA2Warp the odd ones; each acquires the step
    // counter before the first h block it issues.  Measured against three issuers rotating A + W
    // stages: two A issuers beside the W warp won on every shape, profiles/r2_issue_ab.log)
    const int par = warp == 0 ? 0 : 1;
    const bool two = a.issue2 != 0;
    int g = 0;
    for (int t = 0; t < S && (two || par == 0); ++t) {
      const int nkb = kx + (t > 0 ? kh : 0);  // h_{-1} = 0: step 0 has only the x part
      bool waited = false;
      for (int i = 0; i < my_tiles; ++i) {
        const int m0 = tile_m0(i);
        if (a.msync) waited = false;
        for (int j = 0; j < nkb; ++j, ++g) {
          if (two && (g & 1) != par) continue;
          const int s = g % STAGES;
          if (g >= STAGES) wait_sleep(&empty[s], ((g / STAGES) - 1) & 1);
          if (j >= kx && !waited) {
            waited = true;
            // h_{t-1} of this tile's 128 batch rows: wait until every epilogue warp of every tile of
            // the row block (m-tile sync; a.msync = 0: of the whole grid) has released its slice,
            // then order the generic-proxy writes it observed before this thread's async-proxy
            // (TMA) reads
            if (lane == 0) {
              // releases per tile and step: one per epilogue warp (one tile per CTA), one per tile
              // (several tiles per CTA: thousands of same-address releases per step serialised at
              // the L2 -- measured ~6-10 ns each, the whole step time at B = 4096)
              const unsigned per = (unsigned)(a.msync ? a.tiles_n : n_tiles) * (MULTI ? 1u : (unsigned)kREpiWarps);
              const unsigned* ctr = a.counter + (a.msync ? m0 / RBM : 0);
              while (ld_acquire_gpu(ctr) < (unsigned)t * per) {
              }
              fence_proxy_async_global();
              if (trace && t < 64) trace[t * 16 + 0] = rp_gtimer();
              if (mtr && t * my_tiles < 64) mtr[(t * my_tiles) * 16 + 0] = rp_gtimer();
            }
            __syncwarp();
          }
          if (mtr && lane == 0 && j == 0 && t * my_tiles + i < 64) mtr[(t * my_tiles + i) * 16 + 7] = rp_gtimer();
          if (lane == 0) {
            ptx::mbar_arrive_expect_tx(&full[s], R_A_BYTES);
            if (j < kx) {
              ptx::tma_load_2d(&tmX, &full[s], sA + s * R_A_BYTES, j * RBK, t * a.B + m0);
            } else {  // h_{t-1}: one contiguous, pre-swizzled 16 KB block (see hs_index)
              const __nv_bfloat16* src = a.hbuf[(t - 1) & 1] + ((size_t)(kblk(j) - kx) * a.Bp + m0) * RBK;
              ptx::bulk_g2s(sA + s * R_A_BYTES, src, R_A_BYTES, &full[s]);
            }
          }
          __syncwarp();
        }
      }
    }
  } else if (warp == kWWarp) {
    // ---------------- W producer: weights never depend on h ----------------
    if constexpr (WRES) {
      // resident: every packed weight block of this tile, loaded once for the whole sequence
      if (lane == 0) {
        ptx::mbar_arrive_expect_tx(w_full, (uint32_t)(nkw * C::B_BYTES));
        for (int j = 0; j < nkw; ++j) ptx::tma_load_2d(&tmW, w_full, sB + j * C::B_BYTES, j * RBK, tile_n0(0));
      }
    } else {
      // streamed ahead of the barrier in the A ring's stage order
      int g = 0;
      for (int t = 0; t < S; ++t) {
        const int nkb = kx + (t > 0 ? kh : 0);
        for (int i = 0; i < my_tiles; ++i) {
          const int n0 = tile_n0(i);
          for (int j = 0; j < nkb; ++j, ++g) {
            const int s = g % STAGES;
            if (g >= STAGES) wait_sleep(&empty[s], ((g / STAGES) - 1) & 1);
            if (mtr && lane == 0 && j == 0 && t * my_tiles + i < 64) mtr[(t * my_tiles + i) * 16 + 11] = rp_gtimer();
            if (lane == 0) {
              ptx::mbar_arrive_expect_tx(&full[s], C::B_BYTES);
              // packed weight columns: [x part (kx blocks) | h part (kh blocks)] -> column block j
              ptx::tma_load_2d(&tmW, &full[s], sB + s * C::B_BYTES, kblk(j) * RBK, n0);
            }
            __syncwarp();
          }
        }
      }
    }
  } else if (warp == 1) {
    // ---------------- MMA issuer (whole warp, elect.sync issues) ----------------
    constexpr uint32_t idesc = ptx::idesc_bf16(RBM, BN);
    const uint64_t da0 = ptx::desc_sw128(ptx::smem_u32(sA));
    const uint64_t db0 = ptx::desc_sw128(ptx::smem_u32(sB));
    if constexpr (WRES) wait_sleep(w_full, 0);
    int g = 0, u = 0;  // u: work unit (step, tile) counter -> accumulator buffer u & 1
    for (int t = 0; t < S; ++t) {
      const int nkb = kx + (t > 0 ? kh : 0);
      for (int i = 0; i < my_tiles; ++i, ++u) {
        const int buf = u & 1;
        if (u >= 2) wait_sleep(&tempty[buf], ((u >> 1) - 1) & 1);
        ptx::tc_fence_after();
        const uint32_t d = tmem + (uint32_t)(buf * BN);
        for (int j = 0; j < nkb; ++j, ++g) {
          const int s = g % STAGES;
          wait_sleep(&full[s], (g / STAGES) & 1);
          ptx::tc_fence_after();
          if (trace && t < 64 && lane == 0) {
            if (j == 0) trace[t * 16 + 1] = rp_gtimer();
            if (j == kx) trace[t * 16 + 4] = rp_gtimer();  // first h stage landed
          }
          if (mtr && u < 64 && lane == 0) {
            if (j == 0) mtr[u * 16 + 1] = rp_gtimer();
            if (j == kx) mtr[u * 16 + 4] = rp_gtimer();
          }
          const uint64_t da = da0 + (uint64_t)((s * R_A_BYTES) >> 4);
          const uint64_t db = db0 + (uint64_t)(((WRES ? kblk(j) : s) * C::B_BYTES) >> 4);
          if (!(a.dbg & 16))
#pragma unroll
            for (int k = 0; k < RBK / 16; ++k) ptx::umma_bf16_elect(d, da + 2 * k, db + 2 * k, idesc, (j | k) != 0);
          ptx::umma_commit_elect(&empty[s]);
        }
        ptx::umma_commit_elect(&tfull[buf]);
        if (trace && t < 64 && lane == 0) trace[t * 16 + 5] = rp_gtimer();  // last UMMA issued
        if (mtr && u < 64 && lane == 0) mtr[u * 16 + 5] = rp_gtimer();
      }
    }
  } else {
    // ---------------- epilogue: gates, cell, h_t ----------------
    constexpr int U = C::U, UH = C::UH;
    const int q = warp & 3;
    const int half = (warp - 2) >> 2;
    const int H = a.H;
    if constexpr (!MULTI) {
      // one tile for the whole sequence: the recurrent state (LSTM c, GRU h in fp32) stays in
      // registers, and so does the bias for UH <= 16; 128 x 256 tiles (UH = 32) work in chunks of
      // 16 units with the bias read from shared memory (128 accumulator + 128 bias registers would
      // spill)
      constexpr int CU = UH <= 16 ? UH : 16;  // units per chunk
      constexpr int NCH = UH / CU;
      const int row = tile_m0(0) + q * 32 + lane;
      const int unit0 = (tile_n0(0) / BN) * U + half * UH;
      const int nv = min(UH, H - unit0);  // multiple of 8 (H % 8 == 0)
      const bool live = row < a.B && nv > 0;
      float bias[4][NCH == 1 ? UH : 1];
      if constexpr (NCH == 1) {
#pragma unroll
        for (int g = 0; g < 4; ++g)
#pragma unroll
          for (int i = 0; i < UH; ++i) bias[g][i] = s_bias[g * U + half * UH + i];
      }
      float state[UH];  // LSTM: c_{t-1}; GRU: h_{t-1} (fp32)
#pragma unroll
      for (int i = 0; i < UH; ++i) state[i] = 0.0f;
      for (int t = 0; t < S; ++t) {
        const int buf = t & 1;
        wait_sleep(&tfull[buf], (t >> 1) & 1);
        ptx::tc_fence_after();
        if (trace && t < 64 && threadIdx.x == 64) trace[t * 16 + 2] = rp_gtimer();
        const uint32_t tq = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(buf * BN);
#pragma unroll
        for (int ch = 0; ch < NCH; ++ch) {
          float acc[4][CU];
          tmem_ld_gates<CU>(tq + half * UH + ch * CU, U, acc);
          if (ch == NCH - 1) {
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive(&tempty[buf]);  // accumulator buffer free for step t+2
            if (trace && t < 64 && threadIdx.x == 64) trace[t * 16 + 6] = rp_gtimer();  // TMEM read
          }
          float h[CU];
#pragma unroll
          for (int i = 0; i < CU; ++i) {
            float b0, b1, b2, b3;
            if constexpr (NCH == 1) {
              b0 = bias[0][i], b1 = bias[1][i], b2 = bias[2][i], b3 = bias[3][i];
            } else {
              const int c = half * UH + ch * CU + i;
              b0 = s_bias[c], b1 = s_bias[U + c], b2 = s_bias[2 * U + c], b3 = s_bias[3 * U + c];
            }
            h[i] = cell<KIND>(acc[0][i] + b0, acc[1][i] + b1, acc[2][i] + b2, acc[3][i] + b3, state[ch * CU + i]);
          }
          if (live) {
#pragma unroll
            for (int v = 0; v < CU / 8; ++v) {
              const int uo = ch * CU + 8 * v;  // unit offset within this thread's UH units
              if (uo < nv) {
                if (a.seq) store_bf16x8(a.seq + ((size_t)t * a.B + row) * H + unit0 + uo, h + 8 * v);
                if (t == S - 1) store_bf16x8(a.out + (size_t)row * H + unit0 + uo, h + 8 * v);
                else store_bf16x8(a.hbuf[buf] + hs_index(row, unit0 + uo, a.Bp), h + 8 * v);
              }
            }
          }
        }
        if (trace && t < 64 && lane == 0) trace[t * 16 + 6 + warp] = rp_gtimer();  // [8..15] math + stores
        if (t < S - 1) {
          // each warp releases its own slice of h_t (no CTA-wide barrier): the generic-proxy stores
          // are ordered before the release-add by __syncwarp; the consumer acquires the counter and
          // issues fence.proxy.async before its TMA reads
          fence_proxy_async_global();
          if (a.ctarel) {
            // one release per CTA (counting its eight warps): an eighth of the same-address atomics
            // at the counter's L2 slice; bar.sync orders every warp's stores before it (cumulative)
            asm volatile("bar.sync 1, %0;" ::"n"(32 * kREpiWarps) : "memory");
            if (threadIdx.x == 64) red_release_gpu_add(a.counter + (a.msync ? tile_m0(0) / RBM : 0), (unsigned)kREpiWarps);
          } else {
            __syncwarp();
            if (lane == 0) red_release_gpu_add(a.counter + (a.msync ? tile_m0(0) / RBM : 0), 1u);
          }
          if (trace && t < 64 && threadIdx.x == 64) trace[t * 16 + 3] = rp_gtimer();
        }
      }
    } else {
      // several tiles per CTA: with two tiles the recurrent state (LSTM c, GRU h, fp32) stays in
      // registers, one array per tile (its global round trip cost c5's LSTM512 ~4.4 us per step,
      // DESIGN.md "Persistent recurrence"); with more tiles it lives in global memory (LSTM c fp32
      // [B, H]; GRU reads h_{t-1} back in bf16, as the per-step kernel does).  Chunks of 8 units
      // bound the registers.
      // (LSTM only: GRU's bf16 h read-back is cheap, and the extra registers measured slower there)
      constexpr bool kRegs = KIND == EPI_LSTM;
      constexpr int RS = kRegs ? UH : 1;
      const bool regs = kRegs && my_tiles <= 2;
      float rs0[RS], rs1[RS];
#pragma unroll
      for (int k2 = 0; k2 < RS; ++k2) rs0[k2] = rs1[k2] = 0.0f;
      int u = 0;
      for (int t = 0; t < S; ++t) {
        for (int i = 0; i < my_tiles; ++i, ++u) {
          const int buf = u & 1;
          const int row = tile_m0(i) + q * 32 + lane;
          const int n0 = tile_n0(i);
          // the recurrent state of this thread's cells (written by this thread a step ago) is
          // fetched before the accumulator wait, off the epilogue's critical path
          float stp[UH / 8][8];
          {
            const __nv_bfloat16* hprev = a.hbuf[(t - 1) & 1];
#pragma unroll
            for (int c = 0; c < UH / 8; ++c) {
              const int unit = (n0 / BN) * U + half * UH + 8 * c;
              if (regs || t == 0 || row >= a.B || unit >= H) {
#pragma unroll
                for (int e = 0; e < 8; ++e) stp[c][e] = 0.0f;
              } else if constexpr (KIND == EPI_LSTM) {
                const size_t off = (size_t)row * H + unit;
                const float4 c0 = *reinterpret_cast<const float4*>(a.c_state + off);
                const float4 c1 = *reinterpret_cast<const float4*>(a.c_state + off + 4);
                stp[c][0] = c0.x, stp[c][1] = c0.y, stp[c][2] = c0.z, stp[c][3] = c0.w;
                stp[c][4] = c1.x, stp[c][5] = c1.y, stp[c][6] = c1.z, stp[c][7] = c1.w;
              } else {
                const uint4 raw = *reinterpret_cast<const uint4*>(hprev + hs_index(row, unit, a.Bp));
                const __nv_bfloat16* hv = reinterpret_cast<const __nv_bfloat16*>(&raw);
#pragma unroll
                for (int e = 0; e < 8; ++e) stp[c][e] = __bfloat162float(hv[e]);
              }
            }
          }
          wait_sleep(&tfull[buf], (u >> 1) & 1);
          ptx::tc_fence_after();
          if (mtr && u < 64 && threadIdx.x == 64) mtr[u * 16 + 2] = rp_gtimer();
          const uint32_t tq = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(buf * BN);
          // UH <= 16: every chunk's accumulators are read before the buffer is released; UH = 32
          // (bn = 256) reads chunk by chunk (128 live floats would spill) and releases at the end
          constexpr int CH = UH <= 16 ? UH / 8 : 1;
          float acc[UH / 8][4][8];
          auto load_chunk = [&](int c) {  // the four gate blocks of 8 units, one wait
            const uint32_t a0 = tq + half * UH + 8 * c;
            ptx::tmem_ld8x4(a0, a0 + U, a0 + 2 * U, a0 + 3 * U, acc[c]);
          };
          auto release = [&]() {
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive(&tempty[buf]);
            if (mtr && u < 64 && threadIdx.x == 64) mtr[u * 16 + 6] = rp_gtimer();
          };
          if constexpr (CH > 1) {
#pragma unroll
            for (int c = 0; c < UH / 8; ++c) load_chunk(c);
            release();
          }
#pragma unroll
          for (int c = 0; c < UH / 8; ++c) {
            if constexpr (CH == 1) {
              load_chunk(c);
              if (c == UH / 8 - 1) release();
            }
            const int unit = (n0 / BN) * U + half * UH + 8 * c;
            if (row >= a.B || unit >= H) continue;
            const size_t off = (size_t)row * H + unit;
            float st[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) {
              if constexpr (kRegs) st[e] = regs ? (i == 0 ? rs0[8 * c + e] : rs1[8 * c + e]) : stp[c][e];
              else st[e] = stp[c][e];
            }
            const int cb = n0 + half * UH + 8 * c;  // packed bias column of gate block 0
            float h[8];
#pragma unroll
            for (int e = 0; e < 8; ++e)
              h[e] = cell<KIND>(acc[c][0][e] + __ldg(a.bias + cb + e), acc[c][1][e] + __ldg(a.bias + cb + U + e),
                                acc[c][2][e] + __ldg(a.bias + cb + 2 * U + e),
                                acc[c][3][e] + __ldg(a.bias + cb + 3 * U + e), st[e]);
            if (regs) {
              if constexpr (kRegs) {
#pragma unroll
                for (int e = 0; e < 8; ++e) {
                  if (i == 0) rs0[8 * c + e] = st[e];
                  else rs1[8 * c + e] = st[e];
                }
              }
            } else if constexpr (KIND == EPI_LSTM) {
              *reinterpret_cast<float4*>(a.c_state + off) = make_float4(st[0], st[1], st[2], st[3]);
              *reinterpret_cast<float4*>(a.c_state + off + 4) = make_float4(st[4], st[5], st[6], st[7]);
            }
            if (a.seq) store_bf16x8(a.seq + (size_t)t * a.B * H + off, h);
            if (t == S - 1) store_bf16x8(a.out + off, h);
            else store_bf16x8(a.hbuf[t & 1] + hs_index(row, unit, a.Bp), h);
          }
          if (t < S - 1) {
            // the tile's 8 epilogue warps meet at a named barrier; one thread releases the tile
            fence_proxy_async_global();
            asm volatile("bar.sync 1, %0;" ::"n"(32 * kREpiWarps) : "memory");
            if (threadIdx.x == 64) {
              // bar.sync orders the CTA's h stores before this thread's release, which is
              // cumulative at gpu scope (no separate __threadfence)
              red_release_gpu_add(a.counter + (a.msync ? tile_m0(i) / RBM : 0), 1u);
              if (mtr && u < 64) mtr[u * 16 + 3] = rp_gtimer();
            }
          }
        }
      }
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, C::TMEM_COLS);
  }
}

template <int BN, int KIND, bool WRES, bool MULTI>
void launch_rp(const CUtensorMap& tx, const CUtensorMap& th0, const CUtensorMap& th1, const CUtensorMap& tw,
               const RnnPersistArgs& a, int grid, cudaStream_t st) {
  using C = RCfg<BN>;
  auto kern = rnn_persist_kernel<BN, KIND, WRES, MULTI>;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kRSmemBudget));
    attr = true;
  }
  const int smem = a.stages * R_A_BYTES + (WRES ? a.kx + a.kh : a.stages) * C::B_BYTES + C::EXTRA;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kRThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  CK(cudaLaunchKernelEx(&cfg, kern, tx, th0, th1, tw, a));
}

template <int BN, int KIND>
void launch_rp_multi(const CUtensorMap& tx, const CUtensorMap& th0, const CUtensorMap& th1, const CUtensorMap& tw,
                     RnnPersistArgs a, int grid, cudaStream_t st) {
  // several tiles per CTA: W changes per tile, so it is streamed
  a.stages = (192 * 1024) / (R_A_BYTES + RCfg<BN>::B_BYTES);
  if (a.stages > 10) a.stages = 10;
  return launch_rp<BN, KIND, false, true>(tx, th0, th1, tw, a, grid, st);
}

template <int BN, int KIND>
void launch_rp_any(const CUtensorMap& tx, const CUtensorMap& th0, const CUtensorMap& th1, const CUtensorMap& tw,
                   RnnPersistArgs a, int grid, cudaStream_t st) {
  const bool multi = a.tiles_n * a.tiles_m > grid;
  if (multi) return launch_rp_multi<BN, KIND>(tx, th0, th1, tw, a, grid, st);
  static const int wres_env = getenv("DUET_RNN_WRES") ? atoi(getenv("DUET_RNN_WRES")) : 1;
  bool wres = false;
  // with two x / h issuers a resident W pays even next to a 4-stage ring (c4's GRU1024: 160 KB of
  // weights); with one, W streams unless >= 6 stages fit (round 1: 7.72 -> 7.54 us only)
  static const int min_res = getenv("DUET_RNN_WRES_MIN") ? atoi(getenv("DUET_RNN_WRES_MIN")) : 4;
  a.stages = rp_plan(BN, a.kx + a.kh, &wres, a.issue2 ? min_res : 6);
  if (wres && !wres_env) {  // streamed W (comparisons)
    wres = false;
    a.stages = (192 * 1024) / (R_A_BYTES + RCfg<BN>::B_BYTES);
    if (a.stages > 10) a.stages = 10;
  }
  // (TMA multicast of the x_t / h blocks across clusters of 2-8 CTAs was measured in round 1 and
  // removed in round 2: h phase -9..-13% only, and clusters of 8 keep c3's two towers from being
  // co-resident, c3 0.38 -> 0.66 ms)
  if (wres) return launch_rp<BN, KIND, true, false>(tx, th0, th1, tw, a, grid, st);
  return launch_rp<BN, KIND, false, false>(tx, th0, th1, tw, a, grid, st);
}


// ------------------------------------------------------------------------------------------------
// CTA-pair variant of the several-tiles-per-CTA recurrence (round 2).  The several-tile steps were
// bound by the bytes each SM can keep in flight: every 64-wide k-block of a 128 x 256 tile moved
// 16 KB of x/h plus 32 KB of packed weights into one SM, 4 stages of 48 KB filled the shared memory,
// and at the measured ~1.6 us L2 round trip under load that capped a k-block at ~0.41 us (tensor
// pipe ~63% of active cycles, tools/rnn_trace_multi.py + ncu, profiles/r2_rnn.md).  Here two CTAs
// of a cluster form one 256 x 256 pair tile (cta_group::2, UMMA M = 256): each CTA loads its own 128
// rows of x/h and HALF of the weight rows, so a k-block costs each SM 16 + 16 KB and the ring holds
// 7 stages.  The leader's MMA warp issues for both; its commits reach both CTAs' barriers (stage
// free, accumulator ready); both epilogues read their own TMEM (128 rows x all 256 gate columns) and
// release the accumulator on the leader's barrier.  Tiles, grid barrier and cell math are the
// several-tile path's.
constexpr int kPBN = 256;
constexpr int kPWBytes = (kPBN / 2) * RBK * 2;  // this CTA's half of a weight k-block: 16 KB

template <int KIND>
__global__ void __launch_bounds__(kRThreads, 1)
    rnn_pair_kernel(const __grid_constant__ CUtensorMap tmX, const __grid_constant__ CUtensorMap tmH0,
                    const __grid_constant__ CUtensorMap tmH1, const __grid_constant__ CUtensorMap tmW,
                    const RnnPersistArgs a) {
  using C = RCfg<kPBN>;
  constexpr int BN = kPBN;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int STAGES = a.stages;
  uint8_t* sA = smem;
  uint8_t* sB = smem + STAGES * R_A_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(sB + STAGES * kPWBytes);
  uint64_t* empty = full + 10;
  uint64_t* tfull = empty + 10;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = ptx::warp_id();
  const int lane = threadIdx.x & 31;
  const int S = a.S, kx = a.kx, kh = a.kh;
  const uint32_t crank = ptx::cluster_ctarank();
  const uint32_t rank = crank & 1;
  const uint32_t leader = crank & ~1u;
  const int pair = (int)blockIdx.x >> 1, n_pairs = (int)gridDim.x >> 1;
  // h k-blocks rotated per pair (both CTAs of a pair load the same order; see rnn_persist_kernel)
  const int hrot = kh > 0 ? (a.hrot * pair) % kh : 0;
  auto kblk = [&](int j) { return j < kx ? j : kx + (j - kx + hrot) % kh; };
  const int n_ptiles = a.tiles_n * (a.tiles_m >> 1);
  const int n_tiles = a.tiles_n * a.tiles_m;  // 128-row CTA tiles (grid-barrier releases per step)
  const int my_tiles = (n_ptiles - 1 - pair) / n_pairs + 1;
  auto tile_n0 = [&](int i) { return ((pair + i * n_pairs) % a.tiles_n) * BN; };
  auto tile_m0 = [&](int i) { return (((pair + i * n_pairs) / a.tiles_n) * 2 + (int)rank) * RBM; };
  // tools/rnn_trace_multi.py stamps (DUET_RNN_DBG=1), as the one-CTA kernel's
  unsigned long long* mtr = (a.dbg & 1) && blockIdx.x < 128 ? g_rp_trace + (size_t)blockIdx.x * 64 * 16 : nullptr;

  if (threadIdx.x == 0) {
    ptx::tma_prefetch(&tmX);
    ptx::tma_prefetch(&tmH0);
    ptx::tma_prefetch(&tmH1);
    ptx::tma_prefetch(&tmW);
    for (int s = 0; s < STAGES; ++s) {
      ptx::mbar_init(&full[s], 2);  // leader: A producer + W producer expect the pair's bytes
      ptx::mbar_init(&empty[s], 1);  // the leader's commit, multicast to both CTAs
    }
    for (int b = 0; b < 2; ++b) {
      ptx::mbar_init(&tfull[b], 1);
      ptx::mbar_init(&tempty[b], 2 * kREpiWarps);  // leader: both CTAs' epilogue warps
    }
    ptx::fence_mbar_init();
  }
  ptx::cluster_sync();  // barrier init visible to the peer before any TMA completes on the leader's
  if (warp == 1) {
    ptx::tmem_alloc_2sm(tmem_slot, C::TMEM_COLS);
    ptx::tmem_relinquish_2sm();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t full_l0 = ptx::mapa(ptx::smem_u32(&full[0]), leader);

  if (warp == 0 || warp == kA2Warp) {
    // ---------------- A producer: own 128 rows of x_t, [grid barrier], h_{t-1} ----------------
    // (a.issue2: warp 0 the even ring stages, kA2Warp the odd ones, as in rnn_persist_kernel)
    const int par = warp == 0 ? 0 : 1;
    const bool two = a.issue2 != 0;
    int g = 0;
    for (int t = 0; t < S && (two || par == 0); ++t) {
      const int nkb = kx + (t > 0 ? kh : 0);
      bool waited = false;
      for (int i = 0; i < my_tiles; ++i) {
        const int m0 = tile_m0(i);
        if (a.msync) waited = false;
        for (int j = 0; j < nkb; ++j, ++g) {
          if (two && (g & 1) != par) continue;
          const int s = g % STAGES;
          if (g >= STAGES) wait_sleep(&empty[s], ((g / STAGES) - 1) & 1);
          if (j >= kx && !waited) {  // this CTA's 128 rows (m-tile sync) or the grid
            waited = true;
            if (lane == 0) {
              const unsigned per = (unsigned)(a.msync ? a.tiles_n : n_tiles);
              const unsigned* ctr = a.counter + (a.msync ? m0 / RBM : 0);
              while (ld_acquire_gpu(ctr) < (unsigned)t * per) {
              }
              fence_proxy_async_global();
              if (mtr && t * my_tiles < 64) mtr[(t * my_tiles) * 16 + 0] = rp_gtimer();
            }
            __syncwarp();
          }
          if (mtr && lane == 0 && j == 0 && t * my_tiles + i < 64) mtr[(t * my_tiles + i) * 16 + 7] = rp_gtimer();
          if (lane == 0) {
            const uint32_t fb = full_l0 + s * 8;
            if (rank == 0) ptx::mbar_arrive_expect_tx_cl(fb, 2 * R_A_BYTES);
            if (j < kx) {
              ptx::tma_load_2d_2sm(&tmX, fb, sA + s * R_A_BYTES, j * RBK, t * a.B + m0);
            } else {  // pre-swizzled 16 KB h block through a SWIZZLE_NONE map (bytes land as stored)
              ptx::tma_load_2d_2sm(((t - 1) & 1) ? &tmH1 : &tmH0, fb, sA + s * R_A_BYTES, 0, (kblk(j) - kx) * a.Bp + m0);
            }
          }
          __syncwarp();
        }
      }
    }
  } else if (warp == kWWarp) {
    // ---------------- W producer: this CTA's half of each weight k-block ----------------
    int g = 0;
    for (int t = 0; t < S; ++t) {
      const int nkb = kx + (t > 0 ? kh : 0);
      for (int i = 0; i < my_tiles; ++i) {
        const int n0 = tile_n0(i);
        for (int j = 0; j < nkb; ++j, ++g) {
          const int s = g % STAGES;
          if (g >= STAGES) wait_sleep(&empty[s], ((g / STAGES) - 1) & 1);
          if (mtr && lane == 0 && j == 0 && t * my_tiles + i < 64) mtr[(t * my_tiles + i) * 16 + 11] = rp_gtimer();
          if (lane == 0) {
            const uint32_t fb = full_l0 + s * 8;
            if (rank == 0) ptx::mbar_arrive_expect_tx_cl(fb, 2 * kPWBytes);
            ptx::tma_load_2d_2sm(&tmW, fb, sB + s * kPWBytes, kblk(j) * RBK, n0 + (int)rank * (BN / 2));
          }
          __syncwarp();
        }
      }
    }
  } else if (warp == 1) {
    // ---------------- MMA issuer: the leader, for the pair ----------------
    if (rank == 0) {
      constexpr uint32_t idesc = ptx::idesc_bf16(2 * RBM, BN);
      const uint64_t da0 = ptx::desc_sw128(ptx::smem_u32(sA));
      const uint64_t db0 = ptx::desc_sw128(ptx::smem_u32(sB));
      int g = 0, u = 0;
      for (int t = 0; t < S; ++t) {
        const int nkb = kx + (t > 0 ? kh : 0);
        for (int i = 0; i < my_tiles; ++i, ++u) {
          const int buf = u & 1;
          if (u >= 2) wait_sleep(&tempty[buf], ((u >> 1) - 1) & 1);
          ptx::tc_fence_after();
          const uint32_t d = tmem + (uint32_t)(buf * BN);
          for (int j = 0; j < nkb; ++j, ++g) {
            const int s = g % STAGES;
            wait_sleep(&full[s], (g / STAGES) & 1);
            ptx::tc_fence_after();
            if (mtr && u < 64 && lane == 0) {
              if (j == 0) mtr[u * 16 + 1] = rp_gtimer();
              if (j == kx) mtr[u * 16 + 4] = rp_gtimer();
            }
            const uint64_t da = da0 + (uint64_t)((s * R_A_BYTES) >> 4);
            const uint64_t db = db0 + (uint64_t)((s * kPWBytes) >> 4);
#pragma unroll
            for (int k = 0; k < RBK / 16; ++k) ptx::umma_bf16_2sm_elect(d, da + 2 * k, db + 2 * k, idesc, (j | k) != 0);
            ptx::umma_commit_2sm_elect(&empty[s], (uint16_t)(3u << leader));
          }
          ptx::umma_commit_2sm_elect(&tfull[buf], (uint16_t)(3u << leader));
          if (mtr && u < 64 && lane == 0) mtr[u * 16 + 5] = rp_gtimer();
        }
      }
    }
  } else {
    // ---------------- epilogue (the several-tile path's, own 128 rows) ----------------
    constexpr int U = C::U, UH = C::UH;
    const int q = warp & 3;
    const int half = (warp - 2) >> 2;
    const int H = a.H;
    const uint32_t tempty_l = ptx::mapa(ptx::smem_u32(&tempty[0]), leader);
    constexpr bool kRegs = KIND == EPI_LSTM;
    constexpr int RS = kRegs ? UH : 1;
    const bool regs = kRegs && my_tiles <= 2;
    float rs0[RS], rs1[RS];
#pragma unroll
    for (int k2 = 0; k2 < RS; ++k2) rs0[k2] = rs1[k2] = 0.0f;
    int u = 0;
    for (int t = 0; t < S; ++t) {
      for (int i = 0; i < my_tiles; ++i, ++u) {
        const int buf = u & 1;
        const int row = tile_m0(i) + q * 32 + lane;
        const int n0 = tile_n0(i);
        float stp[UH / 8][8];
        {
          const __nv_bfloat16* hprev = a.hbuf[(t - 1) & 1];
#pragma unroll
          for (int c = 0; c < UH / 8; ++c) {
            const int unit = (n0 / BN) * U + half * UH + 8 * c;
            if (regs || t == 0 || row >= a.B || unit >= H) {
#pragma unroll
              for (int e = 0; e < 8; ++e) stp[c][e] = 0.0f;
            } else if constexpr (KIND == EPI_LSTM) {
              const size_t off = (size_t)row * H + unit;
              const float4 c0 = *reinterpret_cast<const float4*>(a.c_state + off);
              const float4 c1 = *reinterpret_cast<const float4*>(a.c_state + off + 4);
              stp[c][0] = c0.x, stp[c][1] = c0.y, stp[c][2] = c0.z, stp[c][3] = c0.w;
              stp[c][4] = c1.x, stp[c][5] = c1.y, stp[c][6] = c1.z, stp[c][7] = c1.w;
            } else {
              const uint4 raw = *reinterpret_cast<const uint4*>(hprev + hs_index(row, unit, a.Bp));
              const __nv_bfloat16* hv = reinterpret_cast<const __nv_bfloat16*>(&raw);
#pragma unroll
              for (int e = 0; e < 8; ++e) stp[c][e] = __bfloat162float(hv[e]);
            }
          }
        }
        wait_sleep(&tfull[buf], (u >> 1) & 1);
        ptx::tc_fence_after();
        if (mtr && u < 64 && threadIdx.x == 64) mtr[u * 16 + 2] = rp_gtimer();
        const uint32_t tq = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(buf * BN);
        float acc[UH / 8][4][8];
#pragma unroll
        for (int c = 0; c < UH / 8; ++c) {
          const uint32_t a0 = tq + half * UH + 8 * c;
          ptx::tmem_ld8x4(a0, a0 + U, a0 + 2 * U, a0 + 3 * U, acc[c]);
          if (c == UH / 8 - 1) {  // accumulator buffer read: release it on the leader
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive_cl_relaxed(tempty_l + buf * 8);
            if (mtr && u < 64 && threadIdx.x == 64) mtr[u * 16 + 6] = rp_gtimer();
          }
          const int unit = (n0 / BN) * U + half * UH + 8 * c;
          if (row >= a.B || unit >= H) continue;
          const size_t off = (size_t)row * H + unit;
          float st[8];
#pragma unroll
          for (int e = 0; e < 8; ++e) {
            if constexpr (kRegs) st[e] = regs ? (i == 0 ? rs0[8 * c + e] : rs1[8 * c + e]) : stp[c][e];
            else st[e] = stp[c][e];
          }
          const int cb = n0 + half * UH + 8 * c;  // packed bias column of gate block 0
          float h[8];
#pragma unroll
          for (int e = 0; e < 8; ++e)
            h[e] = cell<KIND>(acc[c][0][e] + __ldg(a.bias + cb + e), acc[c][1][e] + __ldg(a.bias + cb + U + e),
                              acc[c][2][e] + __ldg(a.bias + cb + 2 * U + e),
                              acc[c][3][e] + __ldg(a.bias + cb + 3 * U + e), st[e]);
          if (regs) {
            if constexpr (kRegs) {
#pragma unroll
              for (int e = 0; e < 8; ++e) {
                if (i == 0) rs0[8 * c + e] = st[e];
                else rs1[8 * c + e] = st[e];
              }
            }
          } else if constexpr (KIND == EPI_LSTM) {
            *reinterpret_cast<float4*>(a.c_state + off) = make_float4(st[0], st[1], st[2], st[3]);
            *reinterpret_cast<float4*>(a.c_state + off + 4) = make_float4(st[4], st[5], st[6], st[7]);
          }
          if (a.seq) store_bf16x8(a.seq + (size_t)t * a.B * H + off, h);
          if (t == S - 1) store_bf16x8(a.out + off, h);
          else store_bf16x8(a.hbuf[t & 1] + hs_index(row, unit, a.Bp), h);
        }
        if (t < S - 1) {
          fence_proxy_async_global();
          asm volatile("bar.sync 1, %0;" ::"n"(32 * kREpiWarps) : "memory");
          if (threadIdx.x == 64) {
            red_release_gpu_add(a.counter + (a.msync ? tile_m0(i) / RBM : 0), 1u);
            if (mtr && u < 64) mtr[u * 16 + 3] = rp_gtimer();
          }
        }
      }
    }
  }
  ptx::tc_fence_before();
  ptx::cluster_sync();  // no CTA exits while its peer can still signal its barriers / TMEM
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc_2sm(tmem, C::TMEM_COLS);
  }
}

CUtensorMap rp_map_plain(const void* base, int64_t rows) {
  // [rows, 64] bf16 rows of 128 B, box 128 rows, no swizzle (the h blocks are stored pre-swizzled)
  CUtensorMap m;
  cuuint64_t dims[2] = {64, (cuuint64_t)rows};
  cuuint64_t strides[1] = {128};
  cuuint32_t box[2] = {64, 128};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = tmap_encode_tiled()(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box,
                                   estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) fail(DUET_ECUDA, "rnn_pair: h tensor map (" + std::to_string((int)r) + ")");
  return m;
}

// false (nothing launched) when the device cannot hold grid / 2 co-resident CTA pairs right now
// (e.g. under a profiler that reserves SM resources); the caller then runs the one-CTA kernel
template <int KIND>
bool launch_rp_pair(const CUtensorMap& tx, RnnPersistArgs a, int grid, cudaStream_t st) {
  auto kern = rnn_pair_kernel<KIND>;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kRSmemBudget));
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
    attr = true;
  }
  a.stages = std::min(10, (kRSmemBudget - RCfg<kPBN>::EXTRA) / (R_A_BYTES + kPWBytes));
  const int smem = a.stages * (R_A_BYTES + kPWBytes) + RCfg<kPBN>::EXTRA;
  {
    static int max_clusters = -1;
    if (max_clusters < 0) {
      cudaLaunchConfig_t q{};
      q.gridDim = dim3(grid);
      q.blockDim = dim3(kRThreads);
      q.dynamicSmemBytes = smem;
      cudaLaunchAttribute ca[1];
      ca[0].id = cudaLaunchAttributeClusterDimension;
      ca[0].val.clusterDim.x = 2;
      ca[0].val.clusterDim.y = 1;
      ca[0].val.clusterDim.z = 1;
      q.attrs = ca;
      q.numAttrs = 1;
      int n = 0;
      if (cudaOccupancyMaxActiveClusters(&n, kern, &q) != cudaSuccess) {
        cudaGetLastError();
        n = 0;
      }
      max_clusters = n;
      if (getenv("DUET_RNN_DBG")) fprintf(stderr, "[rnn_pair] max active 2-CTA clusters %d (need %d)\n", n, grid / 2);
    }
    if (max_clusters < grid / 2) return false;
  }
  const int64_t hrows = (int64_t)a.kh * a.Bp;
  const CUtensorMap th0 = rp_map_plain(a.hbuf[0], hrows), th1 = rp_map_plain(a.hbuf[1], hrows);
  const CUtensorMap tw = make_tmap_bf16_2d(a.wcat, a.w_rows, a.w_cols, kPBN / 2);
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kRThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  at[1].id = cudaLaunchAttributeClusterDimension;
  at[1].val.clusterDim.x = 2;
  at[1].val.clusterDim.y = 1;
  at[1].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 2;
  CK(cudaLaunchKernelEx(&cfg, kern, tx, th0, th1, tw, a));
  return true;
}

}  // namespace

bool rnn_pair_ok(int kind, int bn, int B, int tiles_n, int tiles_m, int sms) {
  // DUET_RNN_PAIR: 0 = never, 1 = GRU only, default 2 = GRU and LSTM -- measured against the
  // one-CTA kernel on one box: GRU1024 at B = 4096 571 -> 542 us, GRU512 447 -> 447; LSTM512 503 ->
  // 537 with the grid barrier, 417 -> 406 us once steps synchronise per row block (round 2,
  // DESIGN.md "Persistent recurrence")
  static const int mode = getenv("DUET_RNN_PAIR") ? atoi(getenv("DUET_RNN_PAIR")) : 2;
  if (mode == 0 || (kind == EPI_LSTM && mode == 1)) return false;
  // under Nsight Compute (which exports NV_NSIGHT_INJECTION_TRANSPORT_TYPE / NV_TPS_LAUNCH_TOKEN to
  // the profiled process) the cooperative cluster launch fails with cudaErrorLaunchFailure although
  // 74 pairs are reported co-resident; profiled runs take the one-CTA kernel (same tiles per CTA,
  // DESIGN.md)
  const bool profiled = getenv("NV_NSIGHT_INJECTION_TRANSPORT_TYPE") || getenv("NV_TPS_LAUNCH_TOKEN") ||
                        getenv("CUDA_INJECTION64_PATH");
  if (profiled && mode != 3) return false;
  return bn == kPBN && tiles_m % 2 == 0 && B % 8 == 0 && tiles_n * tiles_m > sms;
}

int rnn_pair_grid(int tiles_n, int tiles_m, int sms) {
  // the fewest pairs with the same most-pair-tiles-per-pair as all SMs (cf. the CTA grid)
  const int pt = tiles_n * (tiles_m / 2), pairs = sms / 2;
  const int per = (pt + pairs - 1) / pairs;
  return 2 * ((pt + per - 1) / per);
}

void rnn_persist(int kind, int bn, const CUtensorMap& tx, const CUtensorMap& th0, const CUtensorMap& th1,
                 const CUtensorMap& tw, const RnnPersistArgs& a_in, int grid, cudaStream_t st) {
  RnnPersistArgs a = a_in;
  if (a.pair) {
    if (kind == EPI_LSTM && launch_rp_pair<EPI_LSTM>(tx, a, grid, st)) return;
    if (kind == EPI_GRU && launch_rp_pair<EPI_GRU>(tx, a, grid, st)) return;
    a.pair = 0;  // not co-resident: the one-CTA several-tile kernel, same grid and tiles per CTA
  }
  if (kind == EPI_LSTM && bn == 64) return launch_rp_any<64, EPI_LSTM>(tx, th0, th1, tw, a, grid, st);
  if (kind == EPI_LSTM && bn == 128) return launch_rp_any<128, EPI_LSTM>(tx, th0, th1, tw, a, grid, st);
  if (kind == EPI_GRU && bn == 64) return launch_rp_any<64, EPI_GRU>(tx, th0, th1, tw, a, grid, st);
  if (kind == EPI_GRU && bn == 128) return launch_rp_any<128, EPI_GRU>(tx, th0, th1, tw, a, grid, st);
  // 128 x 256 tiles (64 units): half the W bytes per FLOP of bn = 128, double-buffered accumulators
  // fill all 512 TMEM columns; one tile per CTA when 128 x 256 tiles fit the SMs (c5's LSTM256),
  // else several
  if (bn == 256 && kind == EPI_LSTM) return launch_rp_any<256, EPI_LSTM>(tx, th0, th1, tw, a, grid, st);
  if (bn == 256 && kind == EPI_GRU) return launch_rp_any<256, EPI_GRU>(tx, th0, th1, tw, a, grid, st);
  fail(DUET_EUNSUPPORTED, "rnn_persist: bn must be 64, 128 or 256");
}

}  // namespace duet

// debug hook for tools/rnn_trace.py (not part of the C ABI in include/duet.h)
extern "C" int duet_debug_rp_trace(unsigned long long* host, int n) {
  if (n > 128 * 64 * 16) n = 128 * 64 * 16;
  return (int)cudaMemcpyFromSymbol(host, duet::g_rp_trace, (size_t)n * sizeof(unsigned long long));
}
