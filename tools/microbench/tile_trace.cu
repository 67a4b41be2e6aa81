// Phase timing of the tile-local fused MLP kernel (scratch, not product).
#define FELIX_TILE_TRACE 1
#include <cstdio>
#include <vector>
#include <algorithm>
#include <cuda.h>
#include <cuda_runtime.h>
#include "../../paper_conf_asplos_zhaosam24_b200/csrc/mlp_tile.cuh"
using namespace felix;
static CUtensorMap mk(const void* p, int rows, int cols, int box) {
  CUtensorMap m; cuuint64_t d[2] = {(cuuint64_t)cols, (cuuint64_t)rows}; cuuint64_t st[1] = {(cuuint64_t)cols * 2};
  cuuint32_t b[2] = {64, (cuuint32_t)box}; cuuint32_t e[2] = {1, 1};
  cuTensorMapEncodeTiled(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void*>(p), d, st, b, e, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return m;
}
void* dz(size_t b) { void* p; cudaMalloc(&p, b); cudaMemset(p, 0, b); return p; }
template <int CG> void launch(int grid, const TileParams& P) {
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension; at[0].val.clusterDim.x = CG; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
  cudaLaunchConfig_t cfg{}; cfg.gridDim = dim3(grid); cfg.blockDim = dim3(tile::THREADS); cfg.dynamicSmemBytes = tile::SMEM_BYTES;
  cfg.attrs = at; cfg.numAttrs = 1;
  cudaLaunchKernelEx(&cfg, mlp_tile_kernel<CG>, P);
}
int main(int argc, char** argv) {
  const int M = argc > 1 ? atoi(argv[1]) : 4096;
  const int CG = argc > 2 ? atoi(argv[2]) : 2;
  const int K0p = 96;
  const int mt = (M + 127) / 128;
  void* phi = dz((size_t)M * K0p * 2);
  void* W1 = dz(512 * K0p * 2); void* W2 = dz(256 * 512 * 2); void* W3 = dz(256 * 256 * 2);
  float* bias = (float*)dz(4096); float* cpart = (float*)dz((size_t)M * 2 * 4); float* dphi = (float*)dz((size_t)M * K0p * 4);
  TileParams P{};
  P.phi_hi = P.phi_lo = mk(phi, M, K0p, 128);
  P.w1_hi = P.w1_lo = mk(W1, 512, K0p, 128 / CG);
  P.w2_hi = P.w2_lo = mk(W2, 256, 512, 128);
  P.w3_hi = P.w3_lo = mk(W3, 256, 256, 128);
  P.w3t_hi = P.w3t_lo = mk(W3, 256, 256, 128);
  P.w2t_hi = P.w2t_lo = mk(W2, 512, 256, 128 / CG);
  P.w1t_hi = P.w1t_lo = mk(W1, K0p, 512, K0p / CG);
  P.b1 = P.b2 = P.b3 = P.w4 = bias;
  P.c_part = cpart; P.dphi = dphi; P.ld = M; P.n = M; P.n_tiles = mt; P.k0p = K0p; P.n_valid = 82;
  P.idesc_128 = ptx::idesc_f16_f32(128 * CG, 128); P.idesc_256 = ptx::idesc_f16_f32(128 * CG, 256); P.idesc_k0p = ptx::idesc_f16_f32(128 * CG, K0p);
  const int grid = std::min(148 / CG, (mt + CG - 1) / CG) * CG;
  P.trace = (unsigned long long*)dz((size_t)grid * 32 * 8);
  cudaFuncSetAttribute(mlp_tile_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, tile::SMEM_BYTES);
  cudaFuncSetAttribute(mlp_tile_kernel<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, tile::SMEM_BYTES);
  auto L = [&]() { if (CG == 2) launch<2>(grid, P); else launch<1>(grid, P); };
  for (int it = 0; it < 3; ++it) L();
  cudaDeviceSynchronize();
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  const int R = 10;
  for (int it = 0; it < R; ++it) L();
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  printf("CG=%d M=%d grid=%d: %.2f us per launch (err=%s)\n", CG, M, grid, ms * 1000 / R, cudaGetErrorString(cudaGetLastError()));
  // one clean traced launch
  cudaMemset(P.trace, 0, (size_t)grid * 32 * 8);
  L();
  cudaDeviceSynchronize();
  std::vector<unsigned long long> h((size_t)grid * 32);
  cudaMemcpy(h.data(), P.trace, h.size() * 8, cudaMemcpyDeviceToHost);
  unsigned long long t0 = ~0ull;
  for (int b = 0; b < grid; ++b) if (h[b * 32 + 16]) t0 = std::min(t0, h[b * 32 + 16]);
  const char* nm[32] = {"mma:start", "mma:phiFull", "mma:F1issued", "mma:F2issued", "mma:B1issued", "mma:d2ready", "mma:B3issued", 0,
                        "epi:z1_0full", "epi:F1done", "epi:z2full", "epi:F2done", "epi:z3full", "epi:F3done", "epi:B1done", "epi:d2full",
                        "prod:start", 0, "prod:allIssued", 0, 0, 0, 0, 0,
                        "epi:B2done", "epi:B3done", "epi:dphiFull", "epi:B4done", 0, 0, 0, 0};
  for (int sl = 0; sl < 32; ++sl) {
    if (!nm[sl]) continue;
    double mn = 1e18, mx = 0, av = 0; int c = 0;
    for (int b = 0; b < grid; ++b) {
      unsigned long long v = h[b * 32 + sl]; if (!v) continue;
      double d = (sl >= 20 && sl <= 22) ? (double)v : (double)(v - t0);
      mn = std::min(mn, d); mx = std::max(mx, d); av += d; ++c;
    }
    if (c) {
      if (sl >= 20 && sl <= 22) printf("%-20s cycles min/avg/max %.0f / %.0f / %.0f  (first tile only: all tiles)\n", nm[sl], mn, av / c, mx);
      else printf("%-20s us min/avg/max %.2f / %.2f / %.2f\n", nm[sl], mn / 1e3, av / c / 1e3, mx / 1e3);
    }
  }
  return 0;
}
