// CTA-pair tcgen05 GEMM (cta_group::2, UMMA 256 x BN x 16) for the MLP / projection GEMMs.
//
//   D[M, N] = act(A[M, K] * W[N, K]^T + bias)     A, W bf16 K-major; fp32 accumulate in TMEM
//
// A cluster of 2 CTAs (same TPC) computes one 256 x BN tile: CTA r loads rows [m0 + 128 r, +128) of
// A and rows [n0 + r BN/2, +BN/2) of W into its own shared memory (TMA, SWIZZLE_128B); both CTAs'
// copies complete on the LEADER's full barrier; the leader's single MMA thread issues
// tcgen05.mma.cta_group::2, which reads A/B halves from both CTAs' shared memory and writes each
// CTA's 128 accumulator rows into that CTA's TMEM; tcgen05.commit multicasts stage-free and
// accumulator-ready to both CTAs.  Versus the single-CTA tile this halves the W bytes each SM
// pulls from L2 per FLOP and doubles the work per MMA instruction.
#include "../common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace duet {

// Phase timestamps per CTA for the micro-benchmarks (ep.dbg & 32): %globaltimer ns at
// 0 entry, 1 after prologue, 2 first TMA issued, 3 first stage landed (MMA thread),
// 4 last MMA commit issued, 5 accumulator ready (epilogue), 6 epilogue stores done, 7 exit;
// 8 TMEM loaded + bias/act applied, 9 smem staged, 10 TMA store issued, 11 store read done (warp 2), 12 after the
// cluster barrier, 13 after the PDL wait, 14 TMEM allocated (warp 1), 15 bias staged (warp 2).
__device__ unsigned long long g_tc2_trace[16 * 4096];

namespace {

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

constexpr int BM2 = 128;  // rows per CTA (256 per pair)
constexpr int kEpiThreads2 = 256;           // 8 epilogue warps
constexpr int kThreads2 = 64 + kEpiThreads2;  // + TMA producer warp + MMA warp
constexpr int BK2 = 64;   // one SWIZZLE_128B atom of K
constexpr int KB2 = 2;    // k-blocks per pipeline stage: halves barrier round trips per FLOP
constexpr int A2_ATOM = BM2 * BK2 * 2;
constexpr int A2_BYTES = KB2 * A2_ATOM;

template <int BN, bool GA = false>
struct Cfg2 {
  static constexpr int BH = BN / 2;  // W rows per CTA
  static constexpr int B_ATOM = BH * BK2 * 2;
  static constexpr int B_BYTES = KB2 * B_ATOM;
  static constexpr int STAGE = A2_BYTES + B_BYTES;
  static constexpr int STAGES = (200 * 1024) / STAGE > 8 ? 8 : (200 * 1024) / STAGE;
  static constexpr int TMEM_COLS = BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : 256;
  // GA: + the CTA's gather row coordinates [128][F] (int32)
  static constexpr int SMEM = STAGES * STAGE + 1024 + 256 + BN * 4 + (GA ? 128 * kGatherMaxF * 4 : 0);
};

// NP > 1: cluster of 2*NP CTAs = NP pairs along N sharing the A rows.  Each A k-block is split
// into NP row slices of 128/NP rows; pair p's CTA r loads slice p of its rows and multicasts it
// to CTA r of every pair, so the cluster reads A from L2 once instead of NP times.  MMA commits go
// to all 2*NP CTAs so a stage is refilled only after every pair consumed it (empty count NP).
//
// GA: A is gathered (the deep tower's gather-concat fused into this GEMM, SURVEY.md §8(a) A4+A5):
// k-block f of row b is the 128-byte embedding row E[f, ids[b, f]] (D = 64 = one SWIZZLE_128B
// atom), fetched by tile::gather4 TMA loads of 4 rows each, issued by all 32 lanes of the producer
// warp from row coordinates f*R + ids[b, f] that the epilogue warps stage in shared memory.
template <int BN, typename OutT, int NP, bool GA = false>
__global__ void __launch_bounds__(kThreads2, 1)
    gemm2_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmW,
                 const __grid_constant__ CUtensorMap tmO, const TcEpilogue ep, int M, int N, int K) {
  using C = Cfg2<BN, GA>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::STAGES * A2_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(sB + C::STAGES * C::B_BYTES);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tmem_full = empty + C::STAGES;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_full + 1);
  float* s_bias = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(full) + 256);
  int* s_rows = reinterpret_cast<int*>(s_bias + BN);  // GA: [128][F] gather row coordinates

  const int warp = ptx::warp_id();
  const int lane = threadIdx.x & 31;
  const bool tr = (ep.dbg & 32) != 0;
  unsigned long long* trace = g_tc2_trace + 16 * ((blockIdx.y * gridDim.x + blockIdx.x) & 4095);
  if (tr && threadIdx.x == 0) trace[0] = gtimer();
  constexpr bool MC = NP > 1;
  constexpr int SLICE = BM2 / NP;  // A rows per multicast slice
  const uint32_t crank = ptx::cluster_ctarank();
  const uint32_t rank = crank & 1;          // rank within the CTA pair
  const int pair = MC ? (int)(crank >> 1) : 0;
  const int tile_n = (int)(blockIdx.x / (2 * NP)) * NP + pair;
  const int n0 = tile_n * BN;
  const int m0 = blockIdx.y * (2 * BM2) + (int)rank * BM2;  // this CTA's rows
  const int nk = (K + KB2 * BK2 - 1) / (KB2 * BK2);  // stages of KB2 k-blocks
  const int npre = nk < C::STAGES ? nk : C::STAGES;  // stages whose W tiles load before the PDL wait

  if (warp == 0 && lane == 0) {
    ptx::tma_prefetch(&tmA);
    ptx::tma_prefetch(&tmW);
    for (int s = 0; s < C::STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], NP);
    }
    ptx::mbar_init(tmem_full, 1);
    ptx::fence_mbar_init();
  }
  // barrier init visible to the peer CTA before any TMA completes on the leader's barriers
  ptx::cluster_sync_relaxed();
  if (tr && threadIdx.x == 0) trace[12] = gtimer();
  const uint32_t full_leader0 = ptx::mapa(ptx::smem_u32(&full[0]), crank & ~1u);
  if (warp == 0 && lane == 0 && !(ep.dbg & 2)) {
    // weights are graph parameters, never written by the previous kernel: their first stages
    // stream in while the previous kernel drains (programmatic dependent launch)
    for (int kb = 0; kb < npre; ++kb) {
      const uint32_t fb = full_leader0 + kb * 8;
      if (rank == 0) ptx::mbar_arrive_expect_tx_cl(fb, 2 * C::STAGE);
      if (tr && kb == 0) trace[2] = gtimer();
#pragma unroll
      for (int h = 0; h < KB2; ++h)
        ptx::tma_load_2d_2sm(&tmW, fb, sB + kb * C::B_BYTES + h * C::B_ATOM, (kb * KB2 + h) * BK2,
                             n0 + (int)rank * C::BH);
    }
  }
  // wait for the previous kernel BEFORE taking tensor memory: a PDL-dependent CTA that holds TMEM
  // while it waits can starve a co-resident kernel of another stream (observed as a hang with
  // two slots)
  ptx::pdl_wait();
  if (tr && threadIdx.x == 0) trace[13] = gtimer();
  // A tiles of the first stages go out right after the wait, overlapping the TMEM allocation; the
  // pair-wide barrier below (instead of __syncthreads) then guarantees that both CTAs hold their
  // TMEM before the leader's MMA warp can pass it (ep.early_a)
  const int na_early = (ep.early_a && !MC && !(ep.dbg & 2)) ? npre : 0;
  if (warp == 0 && lane == 0) {
    for (int kb = 0; kb < na_early; ++kb)
#pragma unroll
      for (int h = 0; h < KB2; ++h)
        ptx::tma_load_2d_2sm(&tmA, full_leader0 + kb * 8, sA + kb * A2_BYTES + h * A2_ATOM, (kb * KB2 + h) * BK2, m0);
  }
  if (warp == 1) {
    ptx::tmem_alloc_2sm(tmem_slot, C::TMEM_COLS);
    ptx::tmem_relinquish_2sm();
    if (tr && lane == 0) trace[14] = gtimer();
  }
  ptx::tc_fence_before();
  // A loads (below) follow this CTA's alloc, so the leader's first full barrier implies both CTAs'
  // TMEM is allocated before the first MMA.  With multicast, a pair receives A slices from the
  // other pairs, so the whole cluster synchronises instead.
  if constexpr (MC) {
    ptx::cluster_sync();
  } else if (na_early) {
    // CTA barrier (orders the TMEM address in smem) + relaxed pair barrier (the peer's allocation
    // happened; tcgen05 fences order it): the .release cluster arrive would wait for the A loads
    __syncthreads();
    ptx::cluster_sync_relaxed();
  } else {
    __syncthreads();
  }
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  if (tr && threadIdx.x == 0) trace[1] = gtimer();
  ptx::pdl_trigger();

  if (GA && warp == 0) {
    // gathered A: wait for the row coordinates, then per stage every lane issues the gather4 loads
    // of its 4 rows (both k-blocks); lane 0 handles the barrier waits, expect-tx and W tiles
    const int F = ep.g_F;
    asm volatile("bar.sync 2, %0;" ::"n"(kEpiThreads2 + 32) : "memory");
    for (int kb = 0; kb < nk; ++kb) {
      const int s = kb % C::STAGES;
      const bool pre = kb < npre && !(ep.dbg & 2);
      const uint32_t fb = full_leader0 + s * 8;
      if (lane == 0) {
        if (kb >= C::STAGES) ptx::mbar_wait(&empty[s], ((kb / C::STAGES) - 1) & 1);
        if (!pre && rank == 0) ptx::mbar_arrive_expect_tx_cl(fb, 2 * C::STAGE);
      }
      __syncwarp();
#pragma unroll
      for (int h = 0; h < KB2; ++h) {
        const int f = kb * KB2 + h;
        // a k-block past the last field (odd F) re-reads field F-1: the matching W k-block is out of
        // bounds (K = 64 F), zero-filled by TMA, so it adds nothing
        const int fc = f < F ? f : F - 1;
        const int* rr = s_rows + (4 * lane) * F + fc;
        ptx::tma_gather4_2sm(&tmA, fb, sA + s * A2_BYTES + h * A2_ATOM + lane * 512, 0, rr[0], rr[F], rr[2 * F],
                             rr[3 * F]);
        if (lane == 0 && !pre)
          ptx::tma_load_2d_2sm(&tmW, fb, sB + s * C::B_BYTES + h * C::B_ATOM, (kb * KB2 + h) * BK2,
                               n0 + (int)rank * C::BH);
      }
    }
  } else if (warp == 0) {
    if (lane == 0) {
      const uint16_t a_mask = (uint16_t)((NP == 4 ? 0x55u : NP == 2 ? 0x5u : 0x1u) << rank);  // CTA r of every pair
      for (int kb = 0; kb < nk; ++kb) {
        const int s = kb % C::STAGES;
        const bool pre = kb < npre && !(ep.dbg & 2);
        if (kb >= C::STAGES) ptx::mbar_wait(&empty[s], ((kb / C::STAGES) - 1) & 1);
        const uint32_t fb = full_leader0 + s * 8;
        if (ep.dbg & 2) {
          if (rank == 0) ptx::mbar_arrive(&full[s]);
          continue;
        }
        if (!pre && rank == 0) ptx::mbar_arrive_expect_tx_cl(fb, 2 * C::STAGE);
        if (kb < na_early) continue;
#pragma unroll
        for (int h = 0; h < KB2; ++h) {
          if (!MC)
            ptx::tma_load_2d_2sm(&tmA, fb, sA + s * A2_BYTES + h * A2_ATOM, (kb * KB2 + h) * BK2, m0);
          else
            ptx::tma_load_2d_2sm_mc(&tmA, &full[s], sA + s * A2_BYTES + h * A2_ATOM + pair * SLICE * 128,
                                    (kb * KB2 + h) * BK2, m0 + pair * SLICE, a_mask);
          if (!pre)
            ptx::tma_load_2d_2sm(&tmW, fb, sB + s * C::B_BYTES + h * C::B_ATOM, (kb * KB2 + h) * BK2,
                                 n0 + (int)rank * C::BH);
        }
      }
    }
  } else if (warp == 1) {
    if (rank == 0) {
      // the whole warp walks the k loop (uniform descriptors); elect.sync issues each UMMA
      constexpr uint32_t idesc = ptx::idesc_bf16(2 * BM2, BN);
      const uint16_t empty_mask = (uint16_t)((1u << (2 * NP)) - 1);
      const uint16_t pair_mask = (uint16_t)(0x3u << (2 * pair));
      const uint64_t da0 = ptx::desc_sw128(ptx::smem_u32(sA));
      const uint64_t db0 = ptx::desc_sw128(ptx::smem_u32(sB));
      for (int kb = 0; kb < nk; ++kb) {
        const int s = kb % C::STAGES;
        ptx::mbar_wait(&full[s], (kb / C::STAGES) & 1);
        ptx::tc_fence_after();
        if (tr && kb == 0 && lane == 0) trace[3] = gtimer();
#pragma unroll
        for (int h = 0; h < KB2; ++h) {
          // descriptor start address is bits [0, 14) in 16-byte units: offsets add directly
          const uint64_t da = da0 + (uint64_t)((s * A2_BYTES + h * A2_ATOM) >> 4);
          const uint64_t db = db0 + (uint64_t)((s * C::B_BYTES + h * C::B_ATOM) >> 4);
#pragma unroll
          for (int k = 0; k < BK2 / 16; ++k)
            if (!(ep.dbg & 1))
              ptx::umma_bf16_2sm_elect(tmem, da + 2 * k, db + 2 * k, idesc, (kb | h | k) != 0);
        }
        ptx::umma_commit_2sm_elect(&empty[s], empty_mask);
      }
      ptx::umma_commit_2sm_elect(tmem_full, pair_mask);
      if (tr && lane == 0) trace[4] = gtimer();
    }
  } else {
    // epilogue warps 2..9: warp w reads TMEM lanes 32 (w % 4) .. +32 (hardware lane-quarter
    // rule); the two warps of a quarter split the columns.  Bias of this tile -> smem first
    // (overlaps the mainloop).
    for (int c = threadIdx.x - 64; c < BN; c += kEpiThreads2) s_bias[c] = (ep.bias && n0 + c < N) ? ep.bias[n0 + c] : 0.0f;
    if constexpr (GA) {
      // row coordinates f*R + ids[b, f] of this CTA's 128 rows (rows >= M read row 0 of table f;
      // their outputs are clipped by the TMA store)
      const int F = ep.g_F;
      for (int i = threadIdx.x - 64; i < 128 * F; i += kEpiThreads2) {
        const int r = i / F, f = i - r * F;
        const int b = m0 + r;
        s_rows[i] = f * ep.g_R + (b < M ? __ldg(ep.g_ids + (size_t)b * F + f) : 0);
      }
      asm volatile("bar.sync 2, %0;" ::"n"(kEpiThreads2 + 32) : "memory");
    }
    asm volatile("bar.sync 1, %0;" ::"n"(kEpiThreads2) : "memory");
    if (tr && warp == 2 && lane == 0) trace[15] = gtimer();
    const int q = warp & 3;
    const int half = (warp - 2) >> 2;
    const int row = m0 + q * 32 + lane;
    ptx::mbar_wait(tmem_full, 0);
    ptx::tc_fence_after();
    if (tr && warp == 2 && lane == 0) trace[5] = gtimer();
    const uint32_t tq = tmem + ((uint32_t)(q * 32) << 16);
    const int act = ep.act;
    constexpr int EB = (int)sizeof(OutT);
    // columns per TMEM round trip = one swizzle span (<= 128 B) of output
    constexpr int CW = (BN / 2) * EB < 128 ? BN / 2 : 128 / EB;
    if (ep.tma_store && !(ep.dbg & 8)) {
      // Stage the warp's 32 x CW sub-tile in swizzled smem (the A stages are idle once the
      // accumulator is complete) and let TMA write whole lines: a direct st.global from this
      // layout touches 32 rows per instruction.
      constexpr int SPAN = CW * EB;  // bytes per staged row: 128, 64 or 32
      constexpr int SW_SHIFT = SPAN == 128 ? 0 : SPAN == 64 ? 1 : 2;  // row bits feeding the XOR
      constexpr int SW_MASK = SPAN / 16 - 1;
      uint8_t* stage_base = sA + (warp - 2) * (2 * 32 * SPAN);
      int buf = 0;
#pragma unroll 1
      for (int c0 = half * (BN / 2); c0 < (half + 1) * (BN / 2); c0 += CW, buf ^= 1) {
        float v[CW];
        if constexpr (CW == 64) {
          ptx::tmem_ld64(tq + c0, v);
        } else {
#pragma unroll
          for (int j = 0; j < CW / 16; ++j) ptx::tmem_ld16(tq + c0 + 16 * j, v + 16 * j);
        }
        bias_act<CW>(v, s_bias + c0, act);
        if (tr && warp == 2 && lane == 0) trace[8] = gtimer();  // after the first use of the TMEM data
        uint8_t* st_row = stage_base + buf * (32 * SPAN) + lane * SPAN;
        if (lane == 0) ptx::bulk_wait_read<1>();  // this buffer's previous store has read smem
        __syncwarp();
#pragma unroll
        for (int u = 0; u < SPAN / 16; ++u) {
          uint4 pk;
          if constexpr (EB == 2) {
            uint32_t w[4];
#pragma unroll
            for (int t = 0; t < 4; ++t) {
              __nv_bfloat162 h2 = __floats2bfloat162_rn(v[u * 8 + 2 * t], v[u * 8 + 2 * t + 1]);
              w[t] = *reinterpret_cast<uint32_t*>(&h2);
            }
            pk = make_uint4(w[0], w[1], w[2], w[3]);
          } else {
            pk = make_uint4(__float_as_uint(v[u * 4]), __float_as_uint(v[u * 4 + 1]), __float_as_uint(v[u * 4 + 2]),
                            __float_as_uint(v[u * 4 + 3]));
          }
          const int slot = u ^ ((lane >> SW_SHIFT) & SW_MASK);
          *reinterpret_cast<uint4*>(st_row + slot * 16) = pk;
        }
        if (tr && warp == 2 && lane == 0) trace[9] = gtimer();
        ptx::fence_async_smem();
        __syncwarp();
        if (lane == 0) {
          ptx::tma_store_2d(&tmO, stage_base + buf * (32 * SPAN), n0 + c0, m0 + q * 32);
          ptx::bulk_commit();
        }
        if (tr && warp == 2 && lane == 0) trace[10] = gtimer();
      }
      // only the staging reads must finish before the CTA exits (the global writes complete on
      // their own and are visible to dependent grids at grid completion)
      if (lane == 0) ptx::bulk_wait_read<0>();
      if (tr && warp == 2 && lane == 0) trace[11] = gtimer();
    } else {
      OutT* out = reinterpret_cast<OutT*>(ep.out) + (size_t)row * ep.ldo;
#pragma unroll 1
      for (int c0 = half * (BN / 2); c0 < (half + 1) * (BN / 2); c0 += CW) {
        if (ep.dbg & 8) break;
        float v[CW];
        if constexpr (CW == 64) {
          ptx::tmem_ld64(tq + c0, v);
        } else {
#pragma unroll
          for (int j = 0; j < CW / 16; ++j) ptx::tmem_ld16(tq + c0 + 16 * j, v + 16 * j);
        }
        if (ep.dbg & 16) continue;
        if (row < M) {
#pragma unroll
          for (int j = 0; j < CW / 16; ++j) {
            const int col0 = n0 + c0 + 16 * j;
            if (col0 < N) {
              bias_act<16>(v + 16 * j, s_bias + c0 + 16 * j, act);
              store_row16_any(out + col0, v + 16 * j, N - col0);
            }
          }
        }
      }
    }
    if (tr && warp == 2 && lane == 0) trace[6] = gtimer();
  }
  ptx::tc_fence_before();
  ptx::cluster_sync_relaxed();  // TMEM reads ordered by the tcgen05 fences
  if (tr && threadIdx.x == 0) trace[7] = gtimer();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc_2sm(tmem, C::TMEM_COLS);
  }
}

template <int BN, typename OutT, int NP>
void launch2(const CUtensorMap& a, const CUtensorMap& w, const TcEpilogue& ep_in, int M, int N, int K, cudaStream_t st) {
  using C = Cfg2<BN>;
  static const bool no_tma_store = getenv("DUET_TMA_STORE") && atoi(getenv("DUET_TMA_STORE")) == 0;
  TcEpilogue ep = ep_in;
  static const int early_a = getenv("DUET_GEMM_EARLY_A") ? atoi(getenv("DUET_GEMM_EARLY_A")) : 0;
  ep.early_a = early_a;  // opt-in: shorter single launch, but measured slower back to back
  CUtensorMap to{};
  constexpr int EB = (int)sizeof(OutT);
  constexpr int SPAN = (BN / 2) * EB < 128 ? (BN / 2) * EB : 128;
  static_assert(2 * 32 * SPAN * 8 <= C::STAGES * A2_BYTES, "TMA-store staging must fit in the A stages");
  ep.tma_store = !no_tma_store && !(ep.dbg & 8) && SPAN >= 32 &&
                 make_tmap_store_2d(&to, ep.out, EB, M, N, ep.ldo, SPAN);
  auto kern = gemm2_kernel<BN, OutT, NP>;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM));
    attr = true;
  }
  const int tn = (N + BN - 1) / BN;
  dim3 grid(2 * NP * ((tn + NP - 1) / NP), (M + 2 * BM2 - 1) / (2 * BM2));
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = dim3(kThreads2);
  cfg.dynamicSmemBytes = C::SMEM;
  cfg.stream = st;
  const bool no_pdl = !pdl_on(true);
  cudaLaunchAttribute attr2[2];
  attr2[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr2[0].val.programmaticStreamSerializationAllowed = no_pdl ? 0 : 1;
  attr2[1].id = cudaLaunchAttributeClusterDimension;
  attr2[1].val.clusterDim.x = 2 * NP;
  attr2[1].val.clusterDim.y = 1;
  attr2[1].val.clusterDim.z = 1;
  cfg.attrs = attr2;
  cfg.numAttrs = 2;
  CK(cudaLaunchKernelEx(&cfg, kern, a, w, to, ep, M, N, K));
}

template <int BN>
void launch2_gather(const CUtensorMap& tE, const CUtensorMap& w, const TcEpilogue& ep_in, int M, int N, int K,
                    cudaStream_t st) {
  using C = Cfg2<BN, true>;
  TcEpilogue ep = ep_in;
  ep.early_a = 0;
  CUtensorMap to{};
  static_assert(2 * 32 * 128 * 8 <= C::STAGES * A2_BYTES, "TMA-store staging must fit in the A stages");
  ep.tma_store = make_tmap_store_2d(&to, ep.out, 2, M, N, ep.ldo, (BN / 2) * 2 < 128 ? (BN / 2) * 2 : 128);
  auto kern = gemm2_kernel<BN, __nv_bfloat16, 1, true>;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM));
    attr = true;
  }
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(2 * ((N + BN - 1) / BN), (M + 2 * BM2 - 1) / (2 * BM2));
  cfg.blockDim = dim3(kThreads2);
  cfg.dynamicSmemBytes = C::SMEM;
  cfg.stream = st;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = pdl_on(true) ? 1 : 0;
  at[1].id = cudaLaunchAttributeClusterDimension;
  at[1].val.clusterDim.x = 2;
  at[1].val.clusterDim.y = 1;
  at[1].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 2;
  CK(cudaLaunchKernelEx(&cfg, kern, tE, w, to, ep, M, N, K));
}

}  // namespace

CUtensorMap make_tmap_gather4(const void* E, int64_t rows) {
  if ((uintptr_t)E & 15) fail(DUET_EUNSUPPORTED, "gather4 table needs a 16-byte aligned base");
  CUtensorMap m;
  cuuint64_t dims[2] = {64, (cuuint64_t)rows};
  cuuint64_t strides[1] = {128};
  cuuint32_t box[2] = {64, 1};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = tmap_encode_tiled()(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(E), dims, strides, box,
                                   estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                                   CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) fail(DUET_ECUDA, "cuTensorMapEncodeTiled (gather4) failed (" + std::to_string((int)r) + ")");
  return m;
}

bool gemm_tc2_gather_ok(int M, int N, int K, int F, int64_t R) {
  // opt-in (DUET_GATHER_FUSE=1): correct, but tile::gather4 moves 512 B per TMA request and the
  // per-SM request rate makes the fused fc1 ~3x slower than gather kernel + GEMM
  static const bool on = getenv("DUET_GATHER_FUSE") && atoi(getenv("DUET_GATHER_FUSE")) == 1;
  return on && M > 128 && K == 64 * F && F >= 1 && F <= kGatherMaxF && N >= 64 && N % 8 == 0 &&
         (int64_t)F * R < (int64_t)INT32_MAX;
}

void gemm_tc2_gather(const CUtensorMap& tE, const CUtensorMap& tw, int M, int N, int K, int bn, const TcEpilogue& ep,
                     cudaStream_t st) {
  switch (bn) {
    case 64: return launch2_gather<64>(tE, tw, ep, M, N, K, st);
    case 128: return launch2_gather<128>(tE, tw, ep, M, N, K, st);
    case 256: return launch2_gather<256>(tE, tw, ep, M, N, K, st);
  }
  fail(DUET_EUNSUPPORTED, "gemm_tc2_gather: bn must be 64, 128 or 256");
}

int tc2_pick_bn(int M, int N, int K, int sms) {
  // Widest tile that still occupies ~80% of the SM pairs (measured on B200):
  // wide tiles cut L2->SMEM traffic per FLOP, but idle SMs cost more when the grid is small.
  (void)K;
  const int tm = (M + 255) / 256;
  const int pairs = sms / 2;
  for (int bn : {256, 128, 64}) {
    if (bn > N && bn > 64) continue;
    if (tm * ((N + bn - 1) / bn) * 5 >= pairs * 4) return bn;
  }
  return 64;
}

int tc2_pick_np(int M, int N, int bn) {
  // pairs per cluster sharing A by multicast (1, 2 or 4); DUET_GEMM_MC overrides
  (void)M;
  static const int env = getenv("DUET_GEMM_MC") ? atoi(getenv("DUET_GEMM_MC")) : -1;
  const int tn = (N + bn - 1) / bn;
  int np = env >= 0 ? env : 1;
  if (np != 1 && np != 2 && np != 4) np = 1;
  while (np > 1 && tn % np) np >>= 1;
  return np;
}

void gemm_tc2_maps(const CUtensorMap& ta, const CUtensorMap& tw, int M, int N, int K, int bn, int np,
                   const TcEpilogue& ep, int out_bf16, cudaStream_t st) {
  // `ta` must have been encoded with box rows 128 / np (A multicast slices)
#define DUET_L2(BNV)                                                                      \
  if (np == 4)                                                                            \
    return out_bf16 ? launch2<BNV, __nv_bfloat16, 4>(ta, tw, ep, M, N, K, st)            \
                    : launch2<BNV, float, 4>(ta, tw, ep, M, N, K, st);                    \
  if (np == 2)                                                                            \
    return out_bf16 ? launch2<BNV, __nv_bfloat16, 2>(ta, tw, ep, M, N, K, st)            \
                    : launch2<BNV, float, 2>(ta, tw, ep, M, N, K, st);                    \
  return out_bf16 ? launch2<BNV, __nv_bfloat16, 1>(ta, tw, ep, M, N, K, st)              \
                  : launch2<BNV, float, 1>(ta, tw, ep, M, N, K, st);
  switch (bn) {
    case 64: DUET_L2(64)
    case 128: DUET_L2(128)
    case 256: DUET_L2(256)
  }
#undef DUET_L2
  fail(DUET_EUNSUPPORTED, "gemm_tc2: bn must be 64, 128 or 256");
}

}  // namespace duet

// debug hook for tools/gemm_trace.py (not part of the C ABI in include/duet.h)
extern "C" int duet_debug_tc2_trace(unsigned long long* host, int n) {
  if (n > 16 * 4096) n = 16 * 4096;
  return (int)cudaMemcpyFromSymbol(host, duet::g_tc2_trace, (size_t)n * sizeof(unsigned long long));
}
