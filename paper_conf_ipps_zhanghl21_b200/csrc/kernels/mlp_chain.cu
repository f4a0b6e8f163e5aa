// Persistent CTA-pair tcgen05 kernel for a chain of linear layers (the deep
// tower's MLP, e.g. c2's 1664 -> 1024 -> 512 -> 256).
//
//   Y_l = act_l(Y_{l-1} W_l^T + b_l),  l = 0 .. L-1,  Y_{-1} = X      (bf16, fp32 accumulate)
//
// One launch runs every layer.  The work items are the 256 x 128 output tiles of all layers in
// order (layer-major, then row block, then column tile); cluster c of the grid (a CTA pair, as in
// gemm_tc2.cu) takes items c, c + G, c + 2G, ...  A tile of layer l > 0 needs every column tile of
// its row block of layer l-1: the producer waits on a per-(layer, row block) counter that each
// epilogue warp of the producing tiles release-increments after its TMA stores complete.  Items
// are claimed in a global order and all clusters are co-resident (cooperative launch), so every
// wait is on an item that an earlier cluster is already computing: no deadlock.
//
// Versus one gemm_tc2 launch per layer this removes the per-layer prologue (barrier init, TMEM
// allocation), the launch/tail gap between layers and lets the next layer's weights stream in
// while the current layer finishes; the accumulator is double-buffered in TMEM so an item's
// epilogue overlaps the next item's mainloop.
//
// Warp roles per CTA: warp 0 TMA producer, warp 1 MMA issuer (pair leader only; warp-convergent,
// elect.sync), warps 2..9 epilogue (TMEM lane quarter w % 4, the two warps of a quarter take one
// 64-column half each; staged in swizzled smem and written by TMA stores).
#include "../common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace duet {

// per-CTA, per-item %globaltimer stamps when MlpChainArgs::dbg (tools/chain_trace.py):
// [cta][item slot][0] entry, [1] dependency satisfied (producer), [2] first stage landed (MMA),
// [3] last UMMA issued, [4] accumulator ready (epilogue warp 2), [5] released (epilogue warp 2)
__device__ unsigned long long g_chain_trace[296 * 4 * 16];

namespace {

__device__ __forceinline__ unsigned long long ch_gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

constexpr int CBM = 128;                 // rows per CTA (256 per pair)
constexpr int CBN = 128;                 // output columns per tile
constexpr int CBH = CBN / 2;             // W rows per CTA
constexpr int CBK = 64;                  // one SWIZZLE_128B atom of K
constexpr int CKB = 2;                   // k-blocks per stage
constexpr int C_A_ATOM = CBM * CBK * 2;  // 16 KB
constexpr int C_B_ATOM = CBH * CBK * 2;  // 8 KB
constexpr int C_STAGE = CKB * (C_A_ATOM + C_B_ATOM);
constexpr int C_STAGES = 3;
constexpr int C_EPI_WARPS = 8;
constexpr int C_THREADS = 64 + 32 * C_EPI_WARPS;
constexpr int C_STAGING = C_EPI_WARPS * 32 * 128;  // one 32 x 64 bf16 sub-tile per epilogue warp
constexpr int C_SMEM = 1024 + C_STAGES * C_STAGE + C_STAGING + 512;

__device__ __forceinline__ unsigned ld_acquire_gpu_c(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned ld_relaxed_gpu_c(const unsigned* p) {
  unsigned v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
// Poll with relaxed loads (ld.acquire compiles to LD + CCTL.IVALL: invalidating L1 on every probe
// slowed this SM's epilogue warps ~4x), then one acquire load once the target is seen.
__device__ __forceinline__ void wait_counter(const unsigned* p, unsigned target) {
  while (ld_relaxed_gpu_c(p) < target) {
  }
  (void)ld_acquire_gpu_c(p);
}
__device__ __forceinline__ void wait_sleep_c(uint64_t* bar, uint32_t parity) {
  const uint32_t addr = ptx::smem_u32(bar);
  while (!ptx::mbar_try_wait(addr, parity)) {
  }
}
__device__ __forceinline__ void red_release_gpu_add_c(unsigned* p, unsigned v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_global_c() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

struct ItemInfo {
  int l, mb, nb;
};
__device__ __forceinline__ ItemInfo item_info(const MlpChainArgs& a, int item) {
  int l = 0;
  while (l + 1 < a.L && item >= a.item0[l + 1]) ++l;
  const int r = item - a.item0[l];
  return {l, r / a.tiles_n[l], r % a.tiles_n[l]};
}

__global__ void __launch_bounds__(C_THREADS, 1)
    mlp_chain_kernel(const __grid_constant__ MlpChainMaps maps, const MlpChainArgs a) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;                                    // [stage][k-block] 128 x 64
  uint8_t* sB = sA + C_STAGES * CKB * C_A_ATOM;          // [stage][k-block] 64 x 64
  uint8_t* sO = sB + C_STAGES * CKB * C_B_ATOM;          // epilogue staging
  uint64_t* full = reinterpret_cast<uint64_t*>(sO + C_STAGING);
  uint64_t* empty = full + C_STAGES;
  uint64_t* tfull = empty + C_STAGES;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = ptx::warp_id();
  const int lane = threadIdx.x & 31;
  const uint32_t crank = ptx::cluster_ctarank();
  const uint32_t rank = crank & 1;
  const int cluster = (int)blockIdx.x >> 1;
  const int n_clusters = (int)gridDim.x >> 1;
  const int n_items = a.item0[a.L];
  unsigned long long* tr = a.dbg ? g_chain_trace + (size_t)blockIdx.x * 64 : nullptr;
  if (tr && threadIdx.x == 0) tr[0] = ch_gtimer();

  if (warp == 0 && lane == 0) {
    for (int l = 0; l < a.L; ++l) {
      ptx::tma_prefetch(&maps.a[l]);
      ptx::tma_prefetch(&maps.w[l]);
      ptx::tma_prefetch(&maps.o[l]);
    }
    for (int s = 0; s < C_STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      ptx::mbar_init(&tfull[b], 1);
      ptx::mbar_init(&tempty[b], 2 * C_EPI_WARPS);  // both CTAs' epilogue warps (leader's barrier)
    }
    ptx::fence_mbar_init();
  }
  if (warp == 1) {
    ptx::tmem_alloc_2sm(tmem_slot, 2 * CBN);
    ptx::tmem_relinquish_2sm();
  }
  ptx::tc_fence_before();
  ptx::cluster_sync();  // barriers initialised and TMEM allocated in both CTAs
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t full_leader0 = ptx::mapa(ptx::smem_u32(&full[0]), crank & ~1u);

  if (warp == 0) {
    if (lane == 0) {
      int g = 0;
      for (int item = cluster; item < n_items; item += n_clusters) {
        const ItemInfo it = item_info(a, item);
        const int K = a.K[it.l];
        const int nk = (K + CKB * CBK - 1) / (CKB * CBK);
        const int m0 = it.mb * (2 * CBM) + (int)rank * CBM;
        const int n0 = it.nb * CBN;
        bool ready = it.l == 0;
        for (int kb = 0; kb < nk; ++kb, ++g) {
          const int s = g % C_STAGES;
          if (g >= C_STAGES) wait_sleep_c(&empty[s], ((g / C_STAGES) - 1) & 1);
          const uint32_t fb = full_leader0 + s * 8;
          if (rank == 0) ptx::mbar_arrive_expect_tx_cl(fb, 2 * C_STAGE);
#pragma unroll
          for (int h = 0; h < CKB; ++h)  // weights first: they never wait on the previous layer
            ptx::tma_load_2d_2sm(&maps.w[it.l], fb, sB + (s * CKB + h) * C_B_ATOM, (kb * CKB + h) * CBK,
                                 n0 + (int)rank * CBH);
          if (!ready) {
            // the row block of the previous layer: every column tile's epilogue warps (2 CTAs x 8)
            const unsigned target = (unsigned)(2 * C_EPI_WARPS * a.tiles_n[it.l - 1]);
            const unsigned* ctr = a.done + (it.l - 1) * a.m_blocks + it.mb;
            wait_counter(ctr, target);
            fence_proxy_async_global_c();
            ready = true;
            const int slot = (item - cluster) / n_clusters;
            if (tr && slot < 4) tr[slot * 16 + 1] = ch_gtimer();
          }
#pragma unroll
          for (int h = 0; h < CKB; ++h)
            ptx::tma_load_2d_2sm(&maps.a[it.l], fb, sA + (s * CKB + h) * C_A_ATOM, (kb * CKB + h) * CBK, m0);
        }
      }
    }
  } else if (warp == 1) {
    if (rank == 0) {
      const uint64_t da0 = ptx::desc_sw128(ptx::smem_u32(sA));
      const uint64_t db0 = ptx::desc_sw128(ptx::smem_u32(sB));
      constexpr uint32_t idesc = ptx::idesc_bf16(2 * CBM, CBN);
      int g = 0, u = 0;
      for (int item = cluster; item < n_items; item += n_clusters, ++u) {
        const ItemInfo it = item_info(a, item);
        const int nk = (a.K[it.l] + CKB * CBK - 1) / (CKB * CBK);
        const int buf = u & 1;
        if (u >= 2) wait_sleep_c(&tempty[buf], ((u >> 1) - 1) & 1);
        ptx::tc_fence_after();
        const uint32_t d = tmem + (uint32_t)(buf * CBN);
        for (int kb = 0; kb < nk; ++kb, ++g) {
          const int s = g % C_STAGES;
          wait_sleep_c(&full[s], (g / C_STAGES) & 1);
          ptx::tc_fence_after();
          if (tr && kb == 0 && u < 4 && lane == 0) tr[u * 16 + 2] = ch_gtimer();
#pragma unroll
          for (int h = 0; h < CKB; ++h) {
            const uint64_t da = da0 + (uint64_t)(((s * CKB + h) * C_A_ATOM) >> 4);
            const uint64_t db = db0 + (uint64_t)(((s * CKB + h) * C_B_ATOM) >> 4);
#pragma unroll
            for (int k = 0; k < CBK / 16; ++k)
              ptx::umma_bf16_2sm_elect(d, da + 2 * k, db + 2 * k, idesc, (kb | h | k) != 0);
          }
          ptx::umma_commit_2sm_elect(&empty[s], 0x3);
        }
        ptx::umma_commit_2sm_elect(&tfull[buf], 0x3);
        if (tr && u < 4 && lane == 0) tr[u * 16 + 3] = ch_gtimer();
      }
    }
  } else {
    const int q = warp & 3;
    const int half = (warp - 2) >> 2;  // 64-column half of the tile
    const int ew = warp - 2;
    uint8_t* stage = sO + ew * (32 * 128);
    int u = 0;
    for (int item = cluster; item < n_items; item += n_clusters, ++u) {
      const ItemInfo it = item_info(a, item);
      const int m0 = it.mb * (2 * CBM) + (int)rank * CBM;
      const int n0 = it.nb * CBN;
      const int buf = u & 1;
      // this item's bias half -> registers (before the accumulator wait)
      const float* bias = a.bias[it.l];
      float bv[64];
#pragma unroll
      for (int i = 0; i < 64; ++i) bv[i] = 0.0f;
      if (bias && !(a.dbg & 8)) {
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          const float4 b4 = __ldg(reinterpret_cast<const float4*>(bias + n0 + half * 64) + i);
          bv[4 * i] = b4.x, bv[4 * i + 1] = b4.y, bv[4 * i + 2] = b4.z, bv[4 * i + 3] = b4.w;
        }
      }
      wait_sleep_c(&tfull[buf], (u >> 1) & 1);
      ptx::tc_fence_after();
      if (tr && u < 4 && warp == 2 && lane == 0) tr[u * 16 + 4] = ch_gtimer();
      float v[64];
      ptx::tmem_ld64(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(buf * CBN + half * 64), v);
      if (tr && u < 4 && warp == 2 && lane == 0) tr[u * 16 + 6] = ch_gtimer();
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0)  // accumulator buffer free (the pair leader's barrier)
        ptx::mbar_arrive_cl_relaxed(ptx::mapa(ptx::smem_u32(&tempty[buf]), crank & ~1u));
      const int act = (a.dbg & 16) ? 0 : a.act[it.l];
      bias_act<64>(v, bv, act);
      if (tr && u < 4 && warp == 2 && lane == 0) tr[u * 16 + 8] = ch_gtimer();  // act applied
      if (lane == 0) ptx::bulk_wait_read<0>();  // the previous item's store has read the staging
      __syncwarp();
      if (tr && u < 4 && warp == 2 && lane == 0) tr[u * 16 + 9] = ch_gtimer();  // staging free
      uint8_t* st_row = stage + lane * 128;
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        uint32_t w[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          __nv_bfloat162 h2 = __floats2bfloat162_rn(v[c * 8 + 2 * t], v[c * 8 + 2 * t + 1]);
          w[t] = *reinterpret_cast<uint32_t*>(&h2);
        }
        if (!(a.dbg & 64))
          *reinterpret_cast<uint4*>(st_row + ((c ^ (lane & 7)) * 16)) = make_uint4(w[0], w[1], w[2], w[3]);
      }
      if (tr && u < 4 && warp == 2 && lane == 0) tr[u * 16 + 10] = ch_gtimer();  // staged (before fence)
      if (!(a.dbg & 128)) ptx::fence_async_smem();
      __syncwarp();
      if (tr && u < 4 && warp == 2 && lane == 0) tr[u * 16 + 7] = ch_gtimer();
      if (lane == 0) {
        ptx::tma_store_2d(&maps.o[it.l], stage, n0 + half * 64, m0 + q * 32);
        ptx::bulk_commit();
        if (it.l + 1 < a.L) {
          // the next layer reads this sub-tile through TMA: complete the writes, then release
          if (!(a.dbg & 4)) ptx::bulk_wait_all();
          if (!(a.dbg & 2)) fence_proxy_async_global_c();
          red_release_gpu_add_c(a.done + it.l * a.m_blocks + it.mb, 1u);
        }
        if (tr && u < 4 && warp == 2) tr[u * 16 + 5] = ch_gtimer();
      }
      __syncwarp();
    }
    if (lane == 0) ptx::bulk_wait_read<0>();
  }
  ptx::tc_fence_before();
  ptx::cluster_sync();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc_2sm(tmem, 2 * CBN);
  }
}

}  // namespace

bool mlp_chain_ok(int M, const int* N, const int* K, int L) {
  if (L < 2 || L > kMlpChainMax || M <= 128) return false;
  for (int l = 0; l < L; ++l)
    if (N[l] % CBN || K[l] % 8) return false;
  return true;
}

void mlp_chain(const MlpChainMaps& maps, MlpChainArgs a, int sms, cudaStream_t st) {
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(mlp_chain_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, C_SMEM));
    attr = true;
  }
  const int m_blocks = a.m_blocks;
  a.item0[0] = 0;
  for (int l = 0; l < a.L; ++l) a.item0[l + 1] = a.item0[l] + m_blocks * a.tiles_n[l];
  const int pairs = std::min(sms / 2, a.item0[a.L]);
  CK(cudaMemsetAsync(a.done, 0, sizeof(unsigned) * a.L * m_blocks, st));
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(2 * pairs);
  cfg.blockDim = dim3(C_THREADS);
  cfg.dynamicSmemBytes = C_SMEM;
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
  CK(cudaLaunchKernelEx(&cfg, mlp_chain_kernel, maps, a));
}

}  // namespace duet

extern "C" int duet_debug_chain_trace(unsigned long long* host, int n) {
  if (n > 296 * 64) n = 296 * 64;
  return (int)cudaMemcpyFromSymbol(host, duet::g_chain_trace, (size_t)n * sizeof(unsigned long long));
}

namespace duet {
CUtensorMap mlp_chain_out_map(void* out, int M, int N) {
  CUtensorMap m{};
  if (!make_tmap_store_2d(&m, out, 2, M, N, N, 128)) fail(DUET_EUNSUPPORTED, "mlp_chain: output map");
  return m;
}

}  // namespace duet
