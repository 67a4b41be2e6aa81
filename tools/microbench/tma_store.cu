// Latency of a TMA tensor store burst (smem -> global) until cp.async.bulk.wait_group 0 returns, as a
// function of bytes per CTA and of the number of CTAs storing at once (scratch, not product).
//   ./tma_store <ctas> <boxes of 128 rows x 64 fp16 (16 KB) per CTA> <reps>
#include <cstdio>
#include <cstdlib>
#include <cuda.h>
#include <cuda_runtime.h>
#include "../../paper_conf_asplos_zhaosam24_b200/csrc/sm100_ptx.cuh"
using namespace felix;

struct Args { CUtensorMap tm; int boxes, reps; unsigned long long* out; };

__global__ void __launch_bounds__(128, 1) store_burst(const __grid_constant__ Args a) {
  extern __shared__ uint8_t raw[];
  uint8_t* smem = raw + ((1024u - (ptx::smem_u32(raw) & 1023u)) & 1023u);
  for (int i = threadIdx.x; i < a.boxes * 16384 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = i;
  ptx::fence_proxy_async_smem();
  __syncthreads();
  unsigned long long tot = 0, mx = 0;
  for (int r = 0; r < a.reps; ++r) {
    // all CTAs start together (grid-wide arrival counter in out[gridDim.x])
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned long long t0, t1;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
      for (int b = 0; b < a.boxes; ++b) ptx::tma_store_2d(&a.tm, b * 64 % 512, (blockIdx.x * a.boxes + b) / 8 * 128, smem + b * 16384);
      ptx::bulk_commit();
      ptx::bulk_wait<0>();
      asm volatile("fence.proxy.async.global;" ::: "memory");
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
      tot += t1 - t0; mx = t1 - t0 > mx ? t1 - t0 : mx;
    }
    __syncthreads();
    // spacing between bursts so they do not overlap
    if (threadIdx.x == 0) { unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); unsigned long long e = t + 20000; do { asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); } while (t < e); }
  }
  if (threadIdx.x == 0) { a.out[2 * blockIdx.x] = tot / a.reps; a.out[2 * blockIdx.x + 1] = mx; }
}

int main(int argc, char** argv) {
  const int ctas = argc > 1 ? atoi(argv[1]) : 128, boxes = argc > 2 ? atoi(argv[2]) : 2, reps = argc > 3 ? atoi(argv[3]) : 20;
  const int rows = 148 * 16 * 128 / 8, cols = 512;
  void* buf; cudaMalloc(&buf, (size_t)rows * cols * 2);
  Args a{};
  cuuint64_t d[2] = {(cuuint64_t)cols, (cuuint64_t)rows}; cuuint64_t st[1] = {(cuuint64_t)cols * 2};
  cuuint32_t b[2] = {64, 128}; cuuint32_t e[2] = {1, 1};
  cuTensorMapEncodeTiled(&a.tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, buf, d, st, b, e, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  a.boxes = boxes; a.reps = reps;
  cudaMalloc(&a.out, 2 * ctas * 8);
  const int smem = boxes * 16384 + 1024;
  cudaFuncSetAttribute(store_burst, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  store_burst<<<ctas, 128, smem>>>(a);
  cudaDeviceSynchronize();
  unsigned long long h[2 * 148]; cudaMemcpy(h, a.out, 2 * ctas * 8, cudaMemcpyDeviceToHost);
  double avg = 0, mx = 0; for (int i = 0; i < ctas; ++i) { avg += h[2 * i]; mx = h[2 * i + 1] > mx ? h[2 * i + 1] : mx; }
  avg /= ctas;
  printf("ctas=%d bytes/CTA=%d: store->wait_group 0 avg %.2f us, max %.2f us  (%s)\n", ctas, boxes * 16384, avg / 1e3, mx / 1e3,
         cudaGetErrorString(cudaGetLastError()));
  return 0;
}
