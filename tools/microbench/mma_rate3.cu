// tcgen05.mma issue-cost variants (scratch): 3-pass 64-wide K block = 12 MMAs, N=64 (TC floor 48 cyc/MMA)
#include <cstdio>
#include <cuda_runtime.h>
#include "../../paper_conf_asplos_zhaosam24_b200/csrc/sm100_ptx.cuh"
using namespace felix;

__device__ __forceinline__ void mma_elect(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n .reg .pred p, e;\n elect.sync _|e, 0xffffffff;\n setp.ne.b32 p, %4, 0;\n"
               " @e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}"
               :: "r"(d), "l"(a), "l"(b), "r"(idesc), "r"(acc) : "memory");
}

template <int V>
__global__ void __launch_bounds__(128, 1) k_rate(int N, int blocks, unsigned long long* out) {
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
  const uint32_t a_hi = ptx::smem_u32(smem), a_lo = a_hi + 16384, b_hi = ptx::smem_u32(smem + 65536), b_lo = b_hi + 16384;
  if (V == 0) {            // current tile-kernel style: single thread, descriptors built per MMA
    if (threadIdx.x == 0) {
      for (int blk = 0; blk < blocks; ++blk) {
        const uint32_t d = tmem + (blk & 1) * 128;
        for (int kk = 0; kk < 4; ++kk) {
          const uint32_t off = kk * 32;
          ptx::mma_f16_ss(d, ptx::sdesc_k_sw128(a_lo + off), ptx::sdesc_k_sw128(b_hi + off), idesc, (blk || kk) ? 1u : 0u);
          ptx::mma_f16_ss(d, ptx::sdesc_k_sw128(a_hi + off), ptx::sdesc_k_sw128(b_lo + off), idesc, 1u);
          ptx::mma_f16_ss(d, ptx::sdesc_k_sw128(a_hi + off), ptx::sdesc_k_sw128(b_hi + off), idesc, 1u);
        }
      }
      ptx::mma_commit(&bar);
      ptx::mbar_wait(&bar, 0);
    }
  } else if (V == 1) {     // single thread, descriptors precomputed, +2 per K step (16 fp16 = 32 B = 2 x 16 B)
    if (threadIdx.x == 0) {
      const uint64_t dah = ptx::sdesc_k_sw128(a_hi), dal = ptx::sdesc_k_sw128(a_lo), dbh = ptx::sdesc_k_sw128(b_hi), dbl = ptx::sdesc_k_sw128(b_lo);
      for (int blk = 0; blk < blocks; ++blk) {
        const uint32_t d = tmem + (blk & 1) * 128;
#pragma unroll
        for (int kk = 0; kk < 4; ++kk) {
          ptx::mma_f16_ss(d, dal + 2 * kk, dbh + 2 * kk, idesc, (blk || kk) ? 1u : 0u);
          ptx::mma_f16_ss(d, dah + 2 * kk, dbl + 2 * kk, idesc, 1u);
          ptx::mma_f16_ss(d, dah + 2 * kk, dbh + 2 * kk, idesc, 1u);
        }
      }
      ptx::mma_commit(&bar);
      ptx::mbar_wait(&bar, 0);
    }
  } else {                 // whole warp, elect.sync inside the asm, precomputed descriptors
    if (warp == 1) {
      const uint64_t dah = ptx::sdesc_k_sw128(a_hi), dal = ptx::sdesc_k_sw128(a_lo), dbh = ptx::sdesc_k_sw128(b_hi), dbl = ptx::sdesc_k_sw128(b_lo);
      for (int blk = 0; blk < blocks; ++blk) {
        const uint32_t d = tmem + (blk & 1) * 128;
#pragma unroll
        for (int kk = 0; kk < 4; ++kk) {
          mma_elect(d, dal + 2 * kk, dbh + 2 * kk, idesc, (blk || kk) ? 1u : 0u);
          mma_elect(d, dah + 2 * kk, dbl + 2 * kk, idesc, 1u);
          mma_elect(d, dah + 2 * kk, dbh + 2 * kk, idesc, 1u);
        }
      }
      if (threadIdx.x == 32) ptx::mma_commit(&bar);
      __syncwarp();
      ptx::mbar_wait(&bar, 0);
    }
  }
  __syncthreads();
  long long c1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x] = c1 - c0;
  ptx::tc_fence_before(); __syncthreads();
  if (warp == 0) ptx::tmem_dealloc(tmem, 512);
}
template <int V> void run(const char* name, unsigned long long* d) {
  cudaFuncSetAttribute(k_rate<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  for (int N : {64, 128, 256}) {
    const int blocks = 400;
    for (int rep = 0; rep < 2; ++rep) k_rate<V><<<32, 128, 200 * 1024>>>(N, blocks, d);
    cudaDeviceSynchronize();
    unsigned long long h[32]; cudaMemcpy(h, d, 32 * 8, cudaMemcpyDeviceToHost);
    double av = 0; for (int i = 0; i < 32; ++i) av += h[i]; av /= 32;
    printf("%-28s N=%3d: %.1f cycles/MMA (SS floor %d) err=%s\n", name, N, av / (blocks * 12), N / 2 > (128 + N) / 4 ? N / 2 : (128 + N) / 4,
           cudaGetErrorString(cudaGetLastError()));
  }
}
int main() {
  unsigned long long* d; cudaMalloc(&d, 148 * 8);
  run<0>("per-MMA descriptors", d);
  run<1>("precomputed, 1 thread", d);
  run<2>("precomputed, warp+elect", d);
  return 0;
}
