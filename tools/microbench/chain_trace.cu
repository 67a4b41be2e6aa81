// Per-layer phase timing of the persistent MLP chain at C2 size (scratch, not product).
#define FELIX_CHAIN_TRACE 1
#include <cstdio>
#include <vector>
#include <algorithm>
#include <cuda.h>
#include <cuda_runtime.h>
#include "../../paper_conf_asplos_zhaosam24_b200/csrc/mlp_chain.cuh"
using namespace felix;
static CUtensorMap mk(const void* p, int rows, int cols, int box) {
  CUtensorMap m; cuuint64_t d[2] = {(cuuint64_t)cols, (cuuint64_t)rows}; cuuint64_t st[1] = {(cuuint64_t)cols * 2};
  cuuint32_t b[2] = {64, (cuuint32_t)box}; cuuint32_t e[2] = {1, 1};
  cuTensorMapEncodeTiled(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void*>(p), d, st, b, e, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return m;
}
void* dz(size_t b) { void* p; cudaMalloc(&p, b); cudaMemset(p, 0, b); return p; }
int main(int argc, char** argv) {
  const int M = argc > 1 ? atoi(argv[1]) : 4096;
  const int dims[5] = {96, 512, 256, 256, 1};
  const int mt = (M + 127) / 128;
  std::vector<void*> act(4);
  for (int l = 0; l < 4; ++l) act[l] = dz((size_t)M * dims[l] * 2 * 2);   // hi then lo (same buffer twice is fine)
  void* masks[4]; for (int l = 1; l < 3; ++l) masks[l] = dz((size_t)M * dims[l] / 8);
  void* W[4]; void* WT[4]; for (int l = 0; l < 3; ++l) { W[l] = dz((size_t)dims[l + 1] * dims[l] * 2); WT[l] = dz((size_t)dims[l + 1] * dims[l] * 2); }
  float* bias = (float*)dz(4096); float* hw = (float*)dz(4096); float* cpart = (float*)dz((size_t)M * 8 * 4); float* dphi = (float*)dz((size_t)M * 96 * 4 * 4);
  ChainParams P{};
  auto add = [&](int i, int epi, int N, int K, const void* a, const void* w, const void* c, int bn) {
    ChainLayer& L = P.layer[i];
    L.a_hi = L.a_lo = mk(a, M, K, 128); L.b_hi = L.b_lo = mk(w, N, K, bn); L.c_hi = L.c_lo = mk(c, M, N, 128);
    GemmArgs& g = L.args; g.M = M; g.N = N; g.K = K; g.bias = bias; g.head_w = hw; g.c_part = cpart; g.ld_c = M;
    g.out_f32 = dphi; g.out_hi = g.out_lo = (__half*)const_cast<void*>(c); g.ld_out = N; g.ld_f32 = M; g.n_valid = 82; g.ld_mask = (mt * 128); g.mask_out = (uint32_t*)masks[1]; g.mask_in = (const uint32_t*)masks[1];
    L.epi = epi; L.bn = bn; L.ksplit = 1; L.n_tiles_n = N / bn; L.n_tiles = mt * L.n_tiles_n; L.idesc = ptx::idesc_f16_f32(128, bn); L.idesc_cat = ptx::idesc_f16_f32(128, 2 * bn);
  };
  int bnA = argc > 2 ? atoi(argv[2]) : 128, bnB = argc > 3 ? atoi(argv[3]) : 64;
  add(0, EPI_RELU, 512, 96, act[0], W[0], act[1], bnA);
  add(1, EPI_RELU, 256, 512, act[1], W[1], act[2], bnB);
  add(2, EPI_HEAD, 256, 256, act[2], W[2], act[3], bnB);
  add(3, EPI_MASK, 256, 256, act[3], WT[2], act[2], bnB);
  add(4, EPI_MASK, 512, 256, act[2], WT[1], act[1], bnA);
  add(5, EPI_F32T, 96, 512, act[1], WT[0], act[0], argc > 7 ? atoi(argv[7]) : 96);
  // production settings at C2 (felix_api.cu build_plan): exact-mask first backward layer, split-K dL/dphi
  P.layer[2].head_exact = 1; P.layer[3].a_exact = 1;
  P.layer[5].ksplit = argc > 8 ? atoi(argv[8]) : 4;
  {
    const int f32tma = argc > 9 ? atoi(argv[9]) : 1;
    CUtensorMap m; cuuint64_t d[2] = {(cuuint64_t)M, (cuuint64_t)(P.layer[5].ksplit * 96)}; cuuint64_t st[1] = {(cuuint64_t)M * 4};
    cuuint32_t b[2] = {128, (cuuint32_t)P.layer[5].bn}; cuuint32_t e[2] = {1, 1};
    cuTensorMapEncodeTiled(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, dphi, d, st, b, e, CU_TENSOR_MAP_INTERLEAVE_NONE,
                           CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    P.layer[5].c_f32 = m; P.layer[5].f32t_tma = f32tma;
  }
  P.n_layers = 6; P.m_tiles = mt;
  P.grid_bar = (unsigned int*)dz(64);
  int grid = std::min(148, mt * 512 / bnA);
  grid = std::max(grid, std::min(148, mt * P.layer[5].n_tiles_n * P.layer[5].ksplit));
  P.trace = (unsigned long long*)dz((size_t)grid * CHAIN_MAX_LAYERS * 8 * 8 * 2);
  const int CS = argc > 4 ? atoi(argv[4]) : 1;
  const int FLAGS = argc > 5 ? atoi(argv[5]) : 1;       // 1: dataflow flags (CS == 1)
  unsigned int* flags = (unsigned int*)dz((size_t)6 * mt * CHAIN_FLAG_STRIDE * 4);
  int one = 1; int* ep = (int*)dz(4); cudaMemcpy(ep, &one, 4, cudaMemcpyHostToDevice);
  P.flags = FLAGS ? flags : nullptr; P.epoch = ep;
  const int REUSE = argc > 6 ? atoi(argv[6]) : 1;        // 1: own-chunk reuse where the row block is kept
  for (int i = 1; i < 6; ++i)
    P.layer[i].reuse = (FLAGS && REUSE && P.layer[i - 1].epi != EPI_F32T && P.layer[i - 1].n_tiles_n == P.layer[i].n_tiles_n && P.layer[i].ksplit == 1) ? 1 : 0;
  if (CS == 4) grid = std::min(148 / 4, mt) * 4;
  cudaFuncSetAttribute(mlp_chain_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, CHAIN_SMEM_BYTES);
  cudaFuncSetAttribute(mlp_chain_kernel<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, CHAIN_SMEM_BYTES);
  auto launch = [&]() {
    if (FLAGS) cudaMemsetAsync(flags, 0, (size_t)6 * mt * CHAIN_FLAG_STRIDE * 4);
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension; at[0].val.clusterDim.x = CS; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
    cudaLaunchConfig_t cfg{}; cfg.gridDim = dim3(grid); cfg.blockDim = dim3(CHAIN_THREADS); cfg.dynamicSmemBytes = CHAIN_SMEM_BYTES;
    cfg.attrs = at; cfg.numAttrs = 1;
    if (CS == 4) cudaLaunchKernelEx(&cfg, mlp_chain_kernel<4>, P); else cudaLaunchKernelEx(&cfg, mlp_chain_kernel<1>, P);
  };
  for (int it = 0; it < 3; ++it) launch();
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  for (int it = 0; it < 10; ++it) launch();
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  printf("FLAGS=%d CS=%d M=%d grid=%d bnA=%d bnB=%d: %.2f us per chain launch (err=%s)\n", FLAGS, CS, M, grid, bnA, bnB, ms * 100, cudaGetErrorString(cudaGetLastError()));
  std::vector<unsigned long long> h((size_t)grid * CHAIN_MAX_LAYERS * 8), h2((size_t)grid * CHAIN_MAX_LAYERS * 8);
  cudaMemcpy(h.data(), P.trace, h.size() * 8, cudaMemcpyDeviceToHost);
  cudaMemcpy(h2.data(), P.trace + h.size(), h2.size() * 8, cudaMemcpyDeviceToHost);
  unsigned long long t0 = ~0ull;
  for (int b = 0; b < grid; ++b) t0 = std::min(t0, h[(size_t)b * CHAIN_MAX_LAYERS * 8 + 0]);
  const char* nm[7] = {"prodStart", "mma1stFull", "mmaLastCommit", "epiStart", "epiEnd", "flagSeen", "flagRel"};
  for (int l = 0; l < 6; ++l) {
    printf("layer %d:", l);
    for (int sl = 0; sl < 7; ++sl) {
      double mn = 1e18, mx = 0, av = 0; int c = 0;
      for (int b = 0; b < grid; ++b) { unsigned long long v = h[((size_t)b * CHAIN_MAX_LAYERS + l) * 8 + sl]; if (!v) continue; double d = (double)(v - t0); mn = std::min(mn, d); mx = std::max(mx, d); av += d; ++c; }
      if (c) printf("  %s %.2f/%.2f/%.2f", nm[sl], mn / 1e3, av / c / 1e3, mx / 1e3);
    }
    printf("\n");
    printf("   epi chunk0 of tile0:");
    const char* n2[4] = {"bufFree", "tmemLoaded", "smemWritten", "barPassed"};
    for (int sl = 0; sl < 4; ++sl) {
      double av = 0; int c = 0;
      for (int b = 0; b < grid; ++b) { unsigned long long v = h2[((size_t)b * CHAIN_MAX_LAYERS + l) * 8 + sl]; if (!v) continue; av += (double)(v - t0); ++c; }
      if (c) printf("  %s %.2f", n2[sl], av / c / 1e3);
    }
    printf("\n");
  }
  return 0;
}
