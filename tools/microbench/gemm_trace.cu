// Phase timing of one GEMM launch (globaltimer stamps per CTA). Scratch, not product.
#define FELIX_GEMM_TRACE 1
#include <cstdio>
#include <vector>
#include <algorithm>
#include <cuda.h>
#include <cuda_runtime.h>
#include "../../paper_conf_asplos_zhaosam24_b200/csrc/mlp_gemm.cuh"
using namespace felix;
static CUtensorMap mk(const void* p, int rows, int cols, int box) {
  CUtensorMap m; cuuint64_t d[2] = {(cuuint64_t)cols, (cuuint64_t)rows}; cuuint64_t st[1] = {(cuuint64_t)cols * 2};
  cuuint32_t b[2] = {64, (cuuint32_t)box}; cuuint32_t e[2] = {1, 1};
  cuTensorMapEncodeTiled(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void*>(p), d, st, b, e, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return m;
}
template <int BN, int EPI> void run(int M, int N, int K, const char* name) {
  __half *A, *B, *oh, *ol; float *bias, *hw, *cp, *of; uint32_t *mo, *mi;
  cudaMalloc(&A, (size_t)M * K * 2); cudaMalloc(&B, (size_t)N * K * 2); cudaMemset(A, 0, (size_t)M*K*2); cudaMemset(B, 0, (size_t)N*K*2);
  cudaMalloc(&oh, (size_t)M * N * 2); cudaMalloc(&ol, (size_t)M * N * 2); cudaMalloc(&bias, N * 4); cudaMalloc(&hw, N * 4);
  cudaMemset(bias, 0, N*4); cudaMemset(hw, 0, N*4);
  cudaMalloc(&cp, (size_t)M * 8 * 4); cudaMalloc(&of, (size_t)N * M * 4); cudaMalloc(&mo, (size_t)M * N / 8); cudaMalloc(&mi, (size_t)M * N / 8);
  cudaMemset(mi, 0xff, (size_t)M*N/8);
  dim3 grid((M + 127) / 128, N / BN);
  unsigned long long* tr; cudaMalloc(&tr, grid.x * grid.y * 8 * 8); cudaMemset(tr, 0, grid.x*grid.y*64);
  GemmArgs a{}; a.M = M; a.N = N; a.K = K; a.bias = bias; a.head_w = hw; a.out_hi = oh; a.out_lo = ol; a.ld_out = N;
  a.mask_out = mo; a.mask_in = mi; a.c_part = cp; a.ld_c = M; a.out_f32 = of; a.ld_f32 = M; a.n_valid = N; a.trace = tr;
  CUtensorMap ma = mk(A, M, K, 128), mb = mk(B, N, K, BN), mc = mk(oh, M, N, 128);
  int nkb = (K + 63) / 64; int stages = std::min(GemmCfg<BN>::MAX_STAGES, nkb);
  auto kern = mlp_gemm_kernel<BN, EPI>;
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, GemmCfg<BN>::smem_bytes(GemmCfg<BN>::MAX_STAGES));
  for (int it = 0; it < 5; ++it) kern<<<grid, 128, GemmCfg<BN>::smem_bytes(stages)>>>(ma, ma, mb, mb, mc, mc, a, stages);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0); kern<<<grid, 128, GemmCfg<BN>::smem_bytes(stages)>>>(ma, ma, mb, mb, mc, mc, a, stages); cudaEventRecord(e1);
  cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1);
  std::vector<unsigned long long> h(grid.x * grid.y * 8); cudaMemcpy(h.data(), tr, h.size() * 8, cudaMemcpyDeviceToHost);
  unsigned long long t0 = ~0ull, tend = 0; int nb = grid.x * grid.y;
  for (int b = 0; b < nb; ++b) { t0 = std::min(t0, h[b * 8]); tend = std::max(tend, h[b * 8 + 5]); }
  double avg[6] = {0};
  for (int b = 0; b < nb; ++b) for (int s = 0; s < 6; ++s) avg[s] += (double)(h[b * 8 + s] - t0) / nb;
  double mx[6] = {0};
  for (int b = 0; b < nb; ++b) for (int s = 0; s < 6; ++s) mx[s] = std::max(mx[s], (double)(h[b * 8 + s] - t0));
  printf("%-28s grid=%dx%d stages=%d event=%.2fus span=%.2fus | avg ns: start %.0f prolog %.0f firstTMA %.0f mmaDone %.0f epiStart %.0f end %.0f | max: start %.0f end %.0f\n",
         name, grid.x, grid.y, stages, ms * 1e3, (tend - t0) / 1e3, avg[0], avg[1], avg[2], avg[3], avg[4], avg[5], mx[0], mx[5]);
}
int main() {
  run<64, EPI_RELU>(4096, 512, 96, "L1 fwd relu 512x96");
  run<64, EPI_RELU>(4096, 256, 512, "L2 fwd relu 256x512");
  run<64, EPI_HEAD>(4096, 256, 256, "L3 fwd head 256x256");
  run<64, EPI_MASK>(4096, 256, 256, "bwd mask 256x256");
  run<64, EPI_MASK>(4096, 512, 256, "bwd mask 512x256");
  run<96, EPI_F32T>(4096, 96, 512, "dphi f32t 96x512");
  run<128, EPI_RELU>(4096, 512, 96, "L1 BN128");
  run<128, EPI_MASK>(4096, 512, 256, "bwd mask 512 BN128");
  run<64, EPI_RELU>(131072, 512, 96, "C5 L1 fwd");
  run<128, EPI_MASK>(131072, 256, 256, "C5 bwd 256");
  return 0;
}
