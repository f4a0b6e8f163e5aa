// Bisect the fixed cost of the CTA-pair GEMM kernel: nvcc -gencode arch=compute_100a,code=sm_100a
//   -O3 -std=c++17 -I paper_conf_ipps_zhanghl21_b200/csrc tools/cluster_bisect.cu -o /tmp/cb
#include <cstdio>

#include "kernels/kernels.h"
#include "kernels/ptx.cuh"

using namespace duet;

template <int MODE>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(192, 1) k2(int* out) {
  extern __shared__ __align__(1024) uint8_t smem[];
  uint32_t* slot = reinterpret_cast<uint32_t*>(smem);
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem + 64);
  const int warp = threadIdx.x >> 5;
  if (MODE >= 1) {
    if (warp == 0 && threadIdx.x == 0) {
      ptx::mbar_init(bar, 1);
      ptx::fence_mbar_init();
    }
    if (MODE >= 2 && warp == 1) {
      ptx::tmem_alloc_2sm(slot, 256);
      ptx::tmem_relinquish_2sm();
    }
    ptx::tc_fence_before();
    ptx::cluster_sync();
    ptx::tc_fence_after();
    if (MODE >= 3) {
      // leader commits (no MMA) multicast to both CTAs; everyone waits
      if (ptx::cluster_ctarank() == 0 && threadIdx.x == 32) ptx::umma_commit_2sm(bar, 0x3);
      if (warp >= 2) ptx::mbar_wait(bar, 0);
    }
    ptx::tc_fence_before();
    ptx::cluster_sync();
    if (MODE >= 2 && warp == 1) {
      ptx::tc_fence_after();
      ptx::tmem_dealloc_2sm(*slot, 256);
    }
  }
  if (threadIdx.x == 0 && out) out[blockIdx.x] = 1;
}

template <int MODE>
__global__ void __launch_bounds__(192, 1) k1(int* out) {
  extern __shared__ __align__(1024) uint8_t smem[];
  uint32_t* slot = reinterpret_cast<uint32_t*>(smem);
  const int warp = threadIdx.x >> 5;
  if (MODE >= 2 && warp == 1) {
    ptx::tmem_alloc(slot, 256);
    ptx::tmem_relinquish();
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (MODE >= 2 && warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(*slot, 256);
  }
  if (threadIdx.x == 0 && out) out[blockIdx.x] = 1;
}

template <typename F>
float time_graph(F launch, cudaStream_t s) {
  cudaGraph_t g;
  cudaGraphExec_t e;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeRelaxed);
  for (int i = 0; i < 20; ++i) launch();
  cudaStreamEndCapture(s, &g);
  cudaGraphInstantiate(&e, g, 0);
  for (int i = 0; i < 20; ++i) cudaGraphLaunch(e, s);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a, s);
  for (int i = 0; i < 20; ++i) cudaGraphLaunch(e, s);
  cudaEventRecord(b, s);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  cudaError_t err = cudaGetLastError();
  if (err) printf("error %s\n", cudaGetErrorString(err));
  return ms * 1000 / 400;
}

int main() {
  cudaStream_t s;
  cudaStreamCreate(&s);
  int* out;
  cudaMalloc(&out, 4096);
  const int big = 197 * 1024;
  cudaFuncSetAttribute(k2<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(k2<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(k2<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(k2<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(k1<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(k1<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  for (int grid : {16, 64, 148}) {
    for (int smem : {4096, big}) {
      printf("grid %3d smem %6d: k1<0> %6.2f us  k1<2> %6.2f us  k2<0> %6.2f  k2<1> %6.2f  k2<2> %6.2f  k2<3> %6.2f us\n",
             grid, smem, time_graph([&] { k1<0><<<grid, 192, smem, s>>>(out); }, s),
             time_graph([&] { k1<2><<<grid, 192, smem, s>>>(out); }, s),
             time_graph([&] { k2<0><<<grid, 192, smem, s>>>(out); }, s),
             time_graph([&] { k2<1><<<grid, 192, smem, s>>>(out); }, s),
             time_graph([&] { k2<2><<<grid, 192, smem, s>>>(out); }, s),
             time_graph([&] { k2<3><<<grid, 192, smem, s>>>(out); }, s));
    }
  }
  return 0;
}
