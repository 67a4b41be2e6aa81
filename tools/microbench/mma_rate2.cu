// tcgen05.mma SS-mode: which feature of the tile kernel's MMA stream costs throughput (scratch)
#include <cstdio>
#include <cuda_runtime.h>
#include "../../paper_conf_asplos_zhaosam24_b200/csrc/sm100_ptx.cuh"
using namespace felix;
// mode bits: 1 = 3-pass hi/lo addresses, 2 = alternate accumulator halves every 12, 4 = F1 mix (24 x N=64 then 24 x N=128),
//            8 = commit every 12, 16 = accumulate=0 at each block start
__global__ void __launch_bounds__(128, 1) k_rate(int N, int iters, int mode, unsigned long long* out) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) { ptx::mbar_init(&bar, 1); ptx::fence_barrier_init(); }
  if (warp == 0) ptx::tmem_alloc(&slot, 512);
  ptx::tc_fence_before(); __syncthreads(); ptx::tc_fence_after();
  const uint32_t tmem = slot;
  long long c0 = clock64();
  if (threadIdx.x == 0) {
    const uint32_t a_hi = ptx::smem_u32(smem), a_lo = a_hi + 16384, b_hi = ptx::smem_u32(smem + 65536), b_lo = b_hi + 16384;
    int done = 0;
    for (int blk = 0; done < iters; ++blk) {
      int n = N;
      if (mode & 4) n = (blk & 1) ? 128 : 64;
      const uint32_t idesc = ptx::idesc_f16_f32(128, n);
      uint32_t d = tmem;
      if (mode & 2) d += (blk & 1) * 128 + ((blk >> 1) & 1) * 256;
      for (int kk = 0; kk < 4; ++kk) {
        const uint32_t off = kk * 32;
        const uint32_t acc0 = ((mode & 16) && kk == 0) ? 0u : 1u;
        if (mode & 1) {
          ptx::mma_f16_ss(d, ptx::sdesc_k_sw128(a_lo + off), ptx::sdesc_k_sw128(b_hi + off), idesc, acc0);
          ptx::mma_f16_ss(d, ptx::sdesc_k_sw128(a_hi + off), ptx::sdesc_k_sw128(b_lo + off), idesc, 1u);
          ptx::mma_f16_ss(d, ptx::sdesc_k_sw128(a_hi + off), ptx::sdesc_k_sw128(b_hi + off), idesc, 1u);
        } else {
          for (int p = 0; p < 3; ++p)
            ptx::mma_f16_ss(d, ptx::sdesc_k_sw128(a_hi + off), ptx::sdesc_k_sw128(b_hi + off), idesc, (p == 0) ? acc0 : 1u);
        }
      }
      done += 12;
      if (mode & 8) ptx::mma_commit(&bar);
    }
    ptx::mma_commit(&bar);
    // wait for the last phase: count commits
    const int ncommit = ((mode & 8) ? (iters + 11) / 12 : 0) + 1;
    ptx::mbar_wait(&bar, (ncommit - 1) & 1);
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
  const int modes[] = {0, 1, 2, 8, 16, 1 | 2 | 8 | 16, 4, 4 | 1 | 2 | 8 | 16};
  for (int N : {64, 128, 256})
    for (int mode : modes) {
      if ((mode & 4) && N != 128) continue;
      const int iters = 4800;
      for (int rep = 0; rep < 2; ++rep) k_rate<<<32, 128, 200 * 1024>>>(N, iters, mode, d);
      cudaDeviceSynchronize();
      unsigned long long h[32]; cudaMemcpy(h, d, 32 * 8, cudaMemcpyDeviceToHost);
      double av = 0; for (int i = 0; i < 32; ++i) av += h[i]; av /= 32;
      printf("N=%3d mode=%2d: %.1f cycles/MMA  err=%s\n", N, mode, av / iters, cudaGetErrorString(cudaGetLastError()));
    }
  return 0;
}
