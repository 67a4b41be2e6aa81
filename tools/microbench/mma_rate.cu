// tcgen05.mma kind::f16 SS-mode issue-rate microbenchmark (scratch): cycles per MMA (M=128, K=16)
#include <cstdio>
#include <cuda_runtime.h>
#include "../../paper_conf_asplos_zhaosam24_b200/csrc/sm100_ptx.cuh"
using namespace felix;
__global__ void __launch_bounds__(128, 1) k_rate(int N, int iters, int sts, unsigned long long* out) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) { ptx::mbar_init(&bar, 1); ptx::fence_barrier_init(); }
  if (warp == 0) ptx::tmem_alloc(&slot, 512);
  ptx::tc_fence_before(); __syncthreads(); ptx::tc_fence_after();
  const uint32_t tmem = slot;
  const uint32_t idesc = ptx::idesc_f16_f32(128, N);
  long long c0 = clock64();
  if (threadIdx.x == 0) {
    const uint32_t a = ptx::smem_u32(smem), b = ptx::smem_u32(smem + 65536);
    for (int i = 0; i < iters; ++i) {
      const uint32_t off = (i & 3) * 32;
      ptx::mma_f16_ss(tmem, ptx::sdesc_k_sw128(a + off), ptx::sdesc_k_sw128(b + off), idesc, i ? 1u : 0u);
    }
    ptx::mma_commit(&bar);
    ptx::mbar_wait(&bar, 0);
  } else if (sts && warp >= 2) {
    // concurrent generic smem stores (epilogue-like traffic) into a separate region
    uint4* p = reinterpret_cast<uint4*>(smem + 131072);
    for (int i = 0; i < iters * sts; ++i) p[(i * 64 + threadIdx.x) & 4095] = make_uint4(i, i, i, i);
  }
  __syncthreads();
  long long c1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x] = c1 - c0;
  ptx::tc_fence_before(); __syncthreads();
  if (warp == 0) ptx::tmem_dealloc(tmem, 512);
}
int main() {
  unsigned long long* d; cudaMalloc(&d, 148 * 8);
  cudaFuncSetAttribute(k_rate, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  for (int sts : {0, 1, 4})
    for (int N : {64, 96, 128, 256}) {
      const int iters = 4096;
      for (int rep = 0; rep < 2; ++rep) k_rate<<<32, 128, 200 * 1024>>>(N, iters, sts, d);
      cudaDeviceSynchronize();
      unsigned long long h[148]; cudaMemcpy(h, d, 32 * 8, cudaMemcpyDeviceToHost);
      double av = 0; for (int i = 0; i < 32; ++i) av += h[i]; av /= 32;
      printf("sts=%d N=%3d: %.1f cycles/MMA (floor %d)  err=%s\n", sts, N, av / iters, 128 * N / 256, cudaGetErrorString(cudaGetLastError()));
    }
  return 0;
}
