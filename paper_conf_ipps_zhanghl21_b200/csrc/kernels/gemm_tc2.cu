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
constexpr int kThreads2 = 64 + kEpiThreads2 + 32;  // + TMA producer warp + MMA warp + W issuer
// Round 2: the W stream has its own issuing warp (warp kWIss2): one thread's copies complete in issue
// order at ~0.37 us per request, and the single producer issued 2 A + 2 W requests per stage
// (the same finding there).  ep.dbg & 64: one issuer (A/B).
constexpr int kWIss2 = 2 + kEpiThreads2 / 32;
constexpr int BK2 = 64;   // one SWIZZLE_128B atom of K
constexpr int KB2 = 2;    // k-blocks per pipeline stage: halves barrier round trips per FLOP
constexpr int A2_ATOM = BM2 * BK2 * 2;
constexpr int A2_BYTES = KB2 * A2_ATOM;

template <int BN>
struct Cfg2 {
  static constexpr int BH = BN / 2;  // W rows per CTA
  static constexpr int B_ATOM = BH * BK2 * 2;
  static constexpr int B_BYTES = KB2 * B_ATOM;
  static constexpr int STAGE = A2_BYTES + B_BYTES;
  static constexpr int STAGES = (200 * 1024) / STAGE > 8 ? 8 : (200 * 1024) / STAGE;
  static constexpr int TMEM_COLS = BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : 256;
  static constexpr int SMEM = STAGES * STAGE + 1024 + 256 + BN * 4;
};

// (Round 1 also carried A multicast across pairs, a gathered-A variant fusing the deep tower's
// gather-concat, and early A loads before the TMEM allocation -- all correct, all measured slower
// or no faster; removed in round 2.)
template <int BN, typename OutT>
__global__ void __launch_bounds__(kThreads2, 1)
    gemm2_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmW,
                 const __grid_constant__ CUtensorMap tmO, const TcEpilogue ep, int M, int N, int K) {
  using C = Cfg2<BN>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::STAGES * A2_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(sB + C::STAGES * C::B_BYTES);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tmem_full = empty + C::STAGES;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_full + 1);
  float* s_bias = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(full) + 256);

  const int warp = ptx::warp_id();
  const int lane = threadIdx.x & 31;
  const bool tr = (ep.dbg & 32) != 0;
  unsigned long long* trace = g_tc2_trace + 16 * ((blockIdx.y * gridDim.x + blockIdx.x) & 4095);
  if (tr && threadIdx.x == 0) trace[0] = gtimer();
  const uint32_t crank = ptx::cluster_ctarank();
  const uint32_t rank = crank & 1;          // rank within the CTA pair
  const int tile_n = (int)(blockIdx.x / 2);
  const int n0 = tile_n * BN;
  const int m0 = blockIdx.y * (2 * BM2) + (int)rank * BM2;  // this CTA's rows
  const int nk = (K + KB2 * BK2 - 1) / (KB2 * BK2);  // stages of KB2 k-blocks
  const int npre = nk < C::STAGES ? nk : C::STAGES;  // stages whose W tiles load before the PDL wait

  if (warp == 0 && lane == 0) {
    ptx::tma_prefetch(&tmA);
    ptx::tma_prefetch(&tmW);
    for (int s = 0; s < C::STAGES; ++s) {
      ptx::mbar_init(&full[s], (ep.dbg & 64) ? 1 : 2);  // A issuer + W issuer (each the pair's bytes)
      ptx::mbar_init(&empty[s], 1);
    }
    ptx::mbar_init(tmem_full, 1);
    ptx::fence_mbar_init();
  }
  // barrier init visible to the peer CTA before any TMA completes on the leader's barriers
  ptx::cluster_sync_relaxed();
  if (tr && threadIdx.x == 0) trace[12] = gtimer();
  const uint32_t full_leader0 = ptx::mapa(ptx::smem_u32(&full[0]), crank & ~1u);
  const bool split = !(ep.dbg & 64);  // A on warp 0, W on warp kWIss2
  if (warp == (split ? kWIss2 : 0) && lane == 0 && !(ep.dbg & 2)) {
    // weights are graph parameters, never written by the previous kernel: their first stages
    // stream in while the previous kernel drains (programmatic dependent launch)
    for (int kb = 0; kb < npre; ++kb) {
      const uint32_t fb = full_leader0 + kb * 8;
      if (rank == 0) ptx::mbar_arrive_expect_tx_cl(fb, split ? 2 * C::B_BYTES : 2 * C::STAGE);
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
  if (warp == 1) {
    ptx::tmem_alloc_2sm(tmem_slot, C::TMEM_COLS);
    ptx::tmem_relinquish_2sm();
    if (tr && lane == 0) trace[14] = gtimer();
  }
  ptx::tc_fence_before();
  // A loads (below) follow this CTA's alloc, so the leader's first full barrier implies both CTAs'
  // TMEM is allocated before the first MMA
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  if (tr && threadIdx.x == 0) trace[1] = gtimer();
  ptx::pdl_trigger();

  if (split && (warp == 0 || warp == kWIss2)) {
    // two issuers: warp 0 the A k-blocks of every stage, warp kWIss2 the W k-blocks (after the
    // pre-loaded stages); each arrives on the leader's full barrier with the pair's bytes
    if (lane == 0 && !(ep.dbg & 2)) {
      const bool isA = warp == 0;
      for (int kb = isA ? 0 : npre; kb < nk; ++kb) {
        const int s = kb % C::STAGES;
        if (kb >= C::STAGES) ptx::mbar_wait(&empty[s], ((kb / C::STAGES) - 1) & 1);
        const uint32_t fb = full_leader0 + s * 8;
        if (rank == 0) ptx::mbar_arrive_expect_tx_cl(fb, isA ? 2 * A2_BYTES : 2 * C::B_BYTES);
#pragma unroll
        for (int h = 0; h < KB2; ++h) {
          if (isA)
            ptx::tma_load_2d_2sm(&tmA, fb, sA + s * A2_BYTES + h * A2_ATOM, (kb * KB2 + h) * BK2, m0);
          else
            ptx::tma_load_2d_2sm(&tmW, fb, sB + s * C::B_BYTES + h * C::B_ATOM, (kb * KB2 + h) * BK2,
                                 n0 + (int)rank * C::BH);
        }
      }
    }
  } else if (warp == 0) {
    if (lane == 0) {
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
#pragma unroll
        for (int h = 0; h < KB2; ++h) {
          ptx::tma_load_2d_2sm(&tmA, fb, sA + s * A2_BYTES + h * A2_ATOM, (kb * KB2 + h) * BK2, m0);
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
      const uint16_t empty_mask = 0x3u;
      const uint16_t pair_mask = 0x3u;
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
  } else if (warp == kWIss2) {
    // (single-issuer mode: idle)
  } else {
    // epilogue warps 2..9: warp w reads TMEM lanes 32 (w % 4) .. +32 (hardware lane-quarter
    // rule); the two warps of a quarter split the columns.  Bias of this tile -> smem first
    // (overlaps the mainloop).
    for (int c = threadIdx.x - 64; c < BN; c += kEpiThreads2) s_bias[c] = (ep.bias && n0 + c < N) ? ep.bias[n0 + c] : 0.0f;
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

template <int BN, typename OutT>
void launch2(const CUtensorMap& a, const CUtensorMap& w, const TcEpilogue& ep_in, int M, int N, int K, cudaStream_t st) {
  using C = Cfg2<BN>;
  static const bool no_tma_store = getenv("DUET_TMA_STORE") && atoi(getenv("DUET_TMA_STORE")) == 0;
  TcEpilogue ep = ep_in;
  CUtensorMap to{};
  constexpr int EB = (int)sizeof(OutT);
  constexpr int SPAN = (BN / 2) * EB < 128 ? (BN / 2) * EB : 128;
  static_assert(2 * 32 * SPAN * 8 <= C::STAGES * A2_BYTES, "TMA-store staging must fit in the A stages");
  ep.tma_store = !no_tma_store && !(ep.dbg & 8) && SPAN >= 32 &&
                 make_tmap_store_2d(&to, ep.out, EB, M, N, ep.ldo, SPAN);
  auto kern = gemm2_kernel<BN, OutT>;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM));
    attr = true;
  }
  const int tn = (N + BN - 1) / BN;
  dim3 grid(2 * tn, (M + 2 * BM2 - 1) / (2 * BM2));
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
  attr2[1].val.clusterDim.x = 2;
  attr2[1].val.clusterDim.y = 1;
  attr2[1].val.clusterDim.z = 1;
  cfg.attrs = attr2;
  cfg.numAttrs = 2;
  CK(cudaLaunchKernelEx(&cfg, kern, a, w, to, ep, M, N, K));
}

}  // namespace

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

void gemm_tc2_maps(const CUtensorMap& ta, const CUtensorMap& tw, int M, int N, int K, int bn, const TcEpilogue& ep,
                   int out_bf16, cudaStream_t st) {
  switch (bn) {
    case 64: return out_bf16 ? launch2<64, __nv_bfloat16>(ta, tw, ep, M, N, K, st) : launch2<64, float>(ta, tw, ep, M, N, K, st);
    case 128:
      return out_bf16 ? launch2<128, __nv_bfloat16>(ta, tw, ep, M, N, K, st) : launch2<128, float>(ta, tw, ep, M, N, K, st);
    case 256:
      return out_bf16 ? launch2<256, __nv_bfloat16>(ta, tw, ep, M, N, K, st) : launch2<256, float>(ta, tw, ep, M, N, K, st);
  }
  fail(DUET_EUNSUPPORTED, "gemm_tc2: bn must be 64, 128 or 256");
}

}  // namespace duet

// debug hook for tools/gemm_trace.py (not part of the C ABI in include/duet.h)
extern "C" int duet_debug_tc2_trace(unsigned long long* host, int n) {
  if (n > 16 * 4096) n = 16 * 4096;
  return (int)cudaMemcpyFromSymbol(host, duet::g_tc2_trace, (size_t)n * sizeof(unsigned long long));
}
