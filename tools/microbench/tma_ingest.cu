// Per-SM TMA ingest rate (L2-resident operands -> shared memory) as a function of ring depth and stage
// size, with and without the chain's 3-pass tcgen05 MMAs consuming the stages (scratch, not product).
//   ./tma_ingest <ctas> <stages> <boxes_per_stage> <mma: 0 none, 1 = 3-pass bn=64 on (A hi, A lo, B hi, B lo)>
#include <cstdio>
#include <cstdlib>
#include <cuda.h>
#include <cuda_runtime.h>
#include "../../paper_conf_asplos_zhaosam24_b200/csrc/sm100_ptx.cuh"
using namespace felix;

// wait variants: 0 try_wait loop (sm100_ptx.cuh), 1 test_wait spin, 2 try_wait with a 20 ns suspend hint
template <int W> __device__ __forceinline__ void wait_bar(uint64_t* bar, uint32_t parity) {
  const uint32_t a = ptx::smem_u32(bar);
  uint32_t ok = 0;
  do {
    if constexpr (W == 0)
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(ok) : "r"(a), "r"(parity) : "memory");
    else if constexpr (W == 1)
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(ok) : "r"(a), "r"(parity) : "memory");
    else
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, 20;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(ok) : "r"(a), "r"(parity) : "memory");
  } while (!ok);
}
__constant__ int c_box_rows;
#define BOX_BYTES (c_box_rows * 128)
struct Args { CUtensorMap tm; CUtensorMap tm3; CUtensorMap tmB; CUtensorMap tmA4; CUtensorMap tmB4; int mode; int stages, boxes, iters, mma, rows; unsigned long long* out; };

template <int W> __global__ void __launch_bounds__(128, 1) ingest(const __grid_constant__ Args a) {
  extern __shared__ uint8_t raw[];
  uint8_t* smem = raw + ((1024u - (ptx::smem_u32(raw) & 1023u)) & 1023u);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + a.stages * a.boxes * BOX_BYTES);
  uint64_t* empty = full + 16;
  uint32_t* slot = reinterpret_cast<uint32_t*>(empty + 16);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < a.stages; ++s) { ptx::mbar_init(&full[s], 1); ptx::mbar_init(&empty[s], 1); }
    ptx::fence_barrier_init();
  }
  if (warp == 1) ptx::tmem_alloc(slot, 128);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *slot;
  unsigned long long t0 = clock64();
  if (warp == 0 && (lane == 0 || a.mode == 1)) {
    const int row_blocks = a.rows / c_box_rows;
    for (int it = 0; it < a.iters; ++it) {
      const int s = it % a.stages;
      if (it >= a.stages) wait_bar<W>(&empty[s], ((it / a.stages) - 1) & 1);
      if (lane == 0) ptx::mbar_arrive_expect_tx(&full[s], a.mode >= 3 ? 49152 : a.boxes * BOX_BYTES);
      if (a.mode == 1) __syncwarp();
      if (a.mode == 3) {        // chain stage: A hi, A lo (128 rows), B hi, B lo (64 rows): 4 x 2-D boxes, 48 KB
        const int k = it % 8, rb = (blockIdx.x * 7 + it) % row_blocks;
        uint8_t* base = smem + (s * a.boxes) * BOX_BYTES;
        ptx::tma_load_2d(base, &a.tm, k * 64, rb * 128, &full[s]);
        ptx::tma_load_2d(base + 16384, &a.tm, k * 64, ((rb + 5) % row_blocks) * 128, &full[s]);
        ptx::tma_load_2d(base + 32768, &a.tmB, k * 64, 64 * (it & 3), &full[s]);
        ptx::tma_load_2d(base + 40960, &a.tmB, k * 64, 64 * (it & 3) + 256, &full[s]);
      } else if (a.mode == 4) { // same bytes as 2 x 3-D boxes (hi / lo planes)
        const int k = it % 8, rb = (blockIdx.x * 7 + it) % (row_blocks / 2);
        uint8_t* base = smem + (s * a.boxes) * BOX_BYTES;
        asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
                     :: "r"(ptx::smem_u32(base)), "l"(reinterpret_cast<uint64_t>(&a.tmA4)), "r"(k * 64), "r"(rb * 128), "r"(0), "r"(ptx::smem_u32(&full[s])) : "memory");
        asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
                     :: "r"(ptx::smem_u32(base + 32768)), "l"(reinterpret_cast<uint64_t>(&a.tmB4)), "r"(k * 64), "r"(64 * (it & 3)), "r"(0), "r"(ptx::smem_u32(&full[s])) : "memory");
      } else if (a.mode == 2) {
        const int rb = (blockIdx.x * 7 + it) % row_blocks;
        asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
                     :: "r"(ptx::smem_u32(smem + (s * a.boxes) * BOX_BYTES)), "l"(reinterpret_cast<uint64_t>(&a.tm3)), "r"(0), "r"(rb * c_box_rows), "r"(0),
                        "r"(ptx::smem_u32(&full[s])) : "memory");
      } else {
        for (int b = 0; b < a.boxes; ++b) {
          if (a.mode == 1 && b != lane) continue;
          const int k = (it * a.boxes + b) % 8, rb = (blockIdx.x * 7 + it + b) % row_blocks;
          ptx::tma_load_2d(smem + (s * a.boxes + b) * BOX_BYTES, &a.tm, k * 64, rb * c_box_rows, &full[s]);
        }
      }
    }
  } else if (warp == 1 && lane == 0) {
    const uint32_t idesc = ptx::idesc_f16_f32(128, 64);
    for (int it = 0; it < a.iters; ++it) {
      const int s = it % a.stages;
      wait_bar<W>(&full[s], (it / a.stages) & 1);
      ptx::tc_fence_after();
      if (a.mma == 2) {         // N-concat: A hi x [B hi | B lo] (N = 128) + A lo x B hi (N = 64)
        const uint32_t ah = ptx::smem_u32(smem + (s * a.boxes) * BOX_BYTES);
        const uint32_t al = ah + 16384, bh = ah + 32768;
        const uint32_t id128 = ptx::idesc_f16_f32(128, 128);
        for (int kk = 0; kk < 4; ++kk) {
          const uint32_t off = kk * 32;
          ptx::mma_f16_ss(tmem, ptx::sdesc_k_sw128(ah + off), ptx::sdesc_k_sw128(bh + off), id128, (it | kk) != 0);
          ptx::mma_f16_ss(tmem, ptx::sdesc_k_sw128(al + off), ptx::sdesc_k_sw128(bh + off), idesc, 1u);
        }
        ptx::mma_commit(&empty[s]);
      } else if (a.mma) {
        // stage = A hi, A lo, B hi(64 rows), B lo(64 rows) laid out in the first boxes (B tiles use half a box)
        const uint32_t ah = ptx::smem_u32(smem + (s * a.boxes) * BOX_BYTES);
        const uint32_t al = ah + BOX_BYTES, bh = ah + 2 * BOX_BYTES, bl = bh + BOX_BYTES / 2;
        for (int kk = 0; kk < 4; ++kk) {
          const uint32_t off = kk * 32;
          ptx::mma_f16_ss(tmem, ptx::sdesc_k_sw128(al + off), ptx::sdesc_k_sw128(bh + off), idesc, (it | kk) != 0);
          ptx::mma_f16_ss(tmem, ptx::sdesc_k_sw128(ah + off), ptx::sdesc_k_sw128(bl + off), idesc, 1u);
          ptx::mma_f16_ss(tmem, ptx::sdesc_k_sw128(ah + off), ptx::sdesc_k_sw128(bh + off), idesc, 1u);
        }
        ptx::mma_commit(&empty[s]);
      } else {
        ptx::mbar_arrive(&empty[s]);
      }
    }
    // drain
    const int it = a.iters - 1;
    wait_bar<W>(&empty[it % a.stages], (it / a.stages) & 1);
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0) a.out[blockIdx.x] = clock64() - t0;
  if (warp == 1) ptx::tmem_dealloc(tmem, 128);
}

int main(int argc, char** argv) {
  const int ctas = argc > 1 ? atoi(argv[1]) : 128, stages = argc > 2 ? atoi(argv[2]) : 2,
            boxes = argc > 3 ? atoi(argv[3]) : 4, mma = argc > 4 ? atoi(argv[4]) : 0;
  const int W = argc > 5 ? atoi(argv[5]) : 0;
  auto kern = W == 0 ? ingest<0> : W == 1 ? ingest<1> : ingest<2>;
  const int box_rows = argc > 6 ? atoi(argv[6]) : 128;
  cudaMemcpyToSymbol(c_box_rows, &box_rows, 4);
  const int rows = 8192, cols = 512;
  void* buf; cudaMalloc(&buf, (size_t)rows * cols * 2); cudaMemset(buf, 0, (size_t)rows * cols * 2);
  Args a{};
  cuuint64_t d[2] = {(cuuint64_t)cols, (cuuint64_t)rows}; cuuint64_t st[1] = {(cuuint64_t)cols * 2};
  cuuint32_t b[2] = {64, (cuuint32_t)box_rows}; cuuint32_t e[2] = {1, 1};
  cuTensorMapEncodeTiled(&a.tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, buf, d, st, b, e, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  {
    cuuint64_t d3[3] = {64, (cuuint64_t)rows, (cuuint64_t)(cols / 64)}; cuuint64_t st3[2] = {(cuuint64_t)cols * 2, 128};
    cuuint32_t b3[3] = {64, (cuuint32_t)box_rows, (cuuint32_t)boxes}; cuuint32_t e3[3] = {1, 1, 1};
    CUresult r = cuTensorMapEncodeTiled(&a.tm3, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 3, buf, d3, st3, b3, e3, CU_TENSOR_MAP_INTERLEAVE_NONE,
                           CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) printf("tm3 encode failed %d\n", (int)r);
  }
  a.mode = argc > 7 ? atoi(argv[7]) : 0;
  {
    cuuint32_t bb[2] = {64, 64};
    cuTensorMapEncodeTiled(&a.tmB, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, buf, d, st, bb, e, CU_TENSOR_MAP_INTERLEAVE_NONE,
                           CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    cuuint64_t d4[3] = {(cuuint64_t)cols, (cuuint64_t)rows / 2, 2}; cuuint64_t st4[2] = {(cuuint64_t)cols * 2, (cuuint64_t)cols * 2 * rows / 2};
    cuuint32_t ba[3] = {64, 128, 2}, bq[3] = {64, 64, 2}; cuuint32_t e4[3] = {1, 1, 1};
    cuTensorMapEncodeTiled(&a.tmA4, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 3, buf, d4, st4, ba, e4, CU_TENSOR_MAP_INTERLEAVE_NONE,
                           CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    cuTensorMapEncodeTiled(&a.tmB4, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 3, buf, d4, st4, bq, e4, CU_TENSOR_MAP_INTERLEAVE_NONE,
                           CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  }
  a.stages = stages; a.boxes = boxes; a.iters = 2048 / boxes; a.mma = mma; a.rows = rows;
  cudaMalloc(&a.out, ctas * 8);
  const int smem = stages * boxes * box_rows * 128 + 1024 + 512;
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  for (int w = 0; w < 2; ++w) kern<<<ctas, 128, smem>>>(a);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  kern<<<ctas, 128, smem>>>(a);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long h[148]; cudaMemcpy(h, a.out, ctas * 8, cudaMemcpyDeviceToHost);
  double avg = 0; for (int i = 0; i < ctas; ++i) avg += h[i]; avg /= ctas;
  const double bytes = (double)a.iters * (a.mode >= 3 ? 49152 : boxes * box_rows * 128);
  printf("mode=%d rows=%d W=%d ctas=%d stages=%d boxes=%d (%d KB/stage, %d KB in flight) mma=%d: %.1f B/clk/SM (clock64), %.1f GB/s/SM, %.2f us  err=%s\n",
         a.mode, box_rows, W, ctas, stages, boxes, boxes * box_rows / 8, stages * boxes * box_rows / 8, mma, bytes / avg, bytes / (ms * 1e-3) / 1e9, ms * 1e3,
         cudaGetErrorString(cudaGetLastError()));
  return 0;
}
