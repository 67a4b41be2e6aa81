// Standalone check of the tcgen05 split-fp16 GEMM (scratch; not part of the product).
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <vector>
#include <random>
#include <algorithm>
#include <cuda.h>
#include <cuda_runtime.h>
#include "../../paper_conf_asplos_zhaosam24_b200/csrc/mlp_gemm.cuh"

using namespace felix;
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d: %s\n", #x, __LINE__, cudaGetErrorString(e)); exit(1);} } while (0)

static CUtensorMap make_map(const void* p, int rows, int cols, int box_rows) {
  CUtensorMap m;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)cols * 2};
  cuuint32_t box[2] = {64, (cuuint32_t)box_rows};
  cuuint32_t es[2] = {1, 1};
  CUresult r = cuTensorMapEncodeTiled(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void*>(p), dims, strides, box, es,
                                      CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                                      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) { printf("encode failed %d\n", (int)r); exit(1); }
  return m;
}

static void split(const std::vector<float>& x, std::vector<__half>& hi, std::vector<__half>& lo) {
  hi.resize(x.size()); lo.resize(x.size());
  for (size_t i = 0; i < x.size(); ++i) { hi[i] = __float2half_rn(x[i]); lo[i] = __float2half_rn(x[i] - __half2float(hi[i])); }
}
template <class T> T* up(const std::vector<T>& v) { T* d; CK(cudaMalloc(&d, v.size() * sizeof(T) + 256)); CK(cudaMemcpy(d, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice)); return d; }

template <int BN, int EPI>
int run(int M, int N, int K, int nvalid) {
  std::mt19937 g(1234 + EPI);
  std::uniform_real_distribution<float> U(-1.f, 1.f);
  std::vector<float> A((size_t)M * K), B((size_t)N * K), bias(N), hw(N);
  for (auto& a : A) a = U(g) * 3.f;
  for (auto& b : B) b = U(g) * 0.1f;
  for (auto& b : bias) b = U(g) * 0.1f;
  for (auto& b : hw) b = U(g) * 0.1f;
  std::vector<uint32_t> mask_in((size_t)M * (N / 32));
  for (auto& w : mask_in) w = g();
  std::vector<__half> Ah, Al, Bh, Bl;
  split(A, Ah, Al); split(B, Bh, Bl);
  __half *dAh = up(Ah), *dAl = up(Al), *dBh = up(Bh), *dBl = up(Bl);
  float* dbias = up(bias); float* dhw = up(hw);
  uint32_t* dmask_in = up(mask_in);
  __half *ohi, *olo; CK(cudaMalloc(&ohi, (size_t)M * N * 2)); CK(cudaMalloc(&olo, (size_t)M * N * 2));
  uint32_t* dmask_out; CK(cudaMalloc(&dmask_out, (size_t)M * (N / 32) * 4));
  float* cpart; CK(cudaMalloc(&cpart, (size_t)(N / BN) * M * 4));
  float* of32; CK(cudaMalloc(&of32, (size_t)N * M * 4));
  GemmArgs a{};
  a.M = M; a.N = N; a.K = K; a.bias = dbias; a.head_w = dhw; a.out_hi = ohi; a.out_lo = olo; a.ld_out = N;
  a.mask_out = dmask_out; a.mask_in = dmask_in; a.c_part = cpart; a.ld_c = M; a.out_f32 = of32; a.ld_f32 = M; a.n_valid = nvalid;
  CUtensorMap mAh = make_map(dAh, M, K, 128), mAl = make_map(dAl, M, K, 128), mBh = make_map(dBh, N, K, BN), mBl = make_map(dBl, N, K, BN), mCh = make_map(ohi, M, N, 128), mCl = make_map(olo, M, N, 128);
  auto kern = mlp_gemm_kernel<BN, EPI>;
  CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, GemmCfg<BN>::smem_bytes(GemmCfg<BN>::MAX_STAGES)));
  dim3 grid((M + 127) / 128, N / BN);
  kern<<<grid, 128, GemmCfg<BN>::smem_bytes(std::min(GemmCfg<BN>::MAX_STAGES,(K+63)/64))>>>(mAh, mAl, mBh, mBl, mCh, mCl, a, std::min(GemmCfg<BN>::MAX_STAGES,(K+63)/64));
  CK(cudaGetLastError());
  CK(cudaDeviceSynchronize());
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  for (int i = 0; i < 20; ++i) kern<<<grid, 128, GemmCfg<BN>::smem_bytes(std::min(GemmCfg<BN>::MAX_STAGES,(K+63)/64))>>>(mAh, mAl, mBh, mBl, mCh, mCl, a, std::min(GemmCfg<BN>::MAX_STAGES,(K+63)/64));
  cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
  float ms; cudaEventElapsedTime(&ms, e0, e1); ms /= 20;

  std::vector<__half> hhi((size_t)M * N), hlo((size_t)M * N);
  std::vector<uint32_t> hmask((size_t)M * (N / 32));
  std::vector<float> hc((size_t)(N / BN) * M), hf((size_t)N * M);
  CK(cudaMemcpy(hhi.data(), ohi, hhi.size() * 2, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(hlo.data(), olo, hlo.size() * 2, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(hmask.data(), dmask_out, hmask.size() * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(hc.data(), cpart, hc.size() * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(hf.data(), of32, hf.size() * 4, cudaMemcpyDeviceToHost));
  double max_err = 0, max_ref = 0; long bad_mask = 0;
  for (int r = 0; r < M; ++r) {
    double head = 0, head_ref = 0;
    for (int n = 0; n < N; ++n) {
      double acc = 0;
      for (int k = 0; k < K; ++k) acc += (double)A[(size_t)r * K + k] * B[(size_t)n * K + k];
      double ref, got;
      if (EPI == EPI_RELU || EPI == EPI_HEAD) {
        double z = acc + bias[n];
        bool on = z > 0;
        bool gon = (hmask[(size_t)r * (N / 32) + n / 32] >> (n % 32)) & 1;
        if (EPI == EPI_RELU && on != gon && fabs(z) > 1e-4) bad_mask++;
        if (EPI == EPI_RELU) ref = on ? z : 0; else { ref = on ? -hw[n] : 0; head_ref += (on ? z : 0) * hw[n]; }
        got = (double)__half2float(hhi[(size_t)r * N + n]) + (double)__half2float(hlo[(size_t)r * N + n]);
        if (fabs(z) < 1e-4) continue;
      } else if (EPI == EPI_MASK) {
        bool on = (mask_in[(size_t)r * (N / 32) + n / 32] >> (n % 32)) & 1;
        ref = on ? acc : 0;
        got = (double)__half2float(hhi[(size_t)r * N + n]) + (double)__half2float(hlo[(size_t)r * N + n]);
      } else {
        if (n >= nvalid) continue;
        ref = acc; got = hf[(size_t)n * M + r];
      }
      max_err = fmax(max_err, fabs(got - ref)); max_ref = fmax(max_ref, fabs(ref));
    }
    if (EPI == EPI_HEAD) {
      for (int t = 0; t < N / BN; ++t) head += hc[(size_t)t * M + r];
      max_err = fmax(max_err, fabs(head - head_ref)); max_ref = fmax(max_ref, fabs(head_ref));
    }
  }
  double flops = 2.0 * M * N * K * 3;
  printf("BN=%d EPI=%d M=%d N=%d K=%d : max_abs_err=%.3e max_ref=%.3e rel=%.3e bad_mask=%ld  %.2f us  %.1f TFLOP/s(3-pass)\n",
         BN, EPI, M, N, K, max_err, max_ref, max_err / max_ref, bad_mask, ms * 1e3, flops / (ms * 1e-3) / 1e12);
  return (max_err / max_ref < 1e-5 && bad_mask == 0) ? 0 : 1;
}

int main() {
  int fails = 0;
  fails += run<128, EPI_RELU>(300, 512, 96, 0);
  fails += run<128, EPI_HEAD>(300, 256, 512, 0);
  fails += run<128, EPI_MASK>(300, 512, 256, 0);
  fails += run<96, EPI_F32T>(300, 96, 512, 82);
  fails += run<64, EPI_RELU>(4096, 256, 512, 0);
  fails += run<256, EPI_HEAD>(4096, 256, 256, 0);
  fails += run<128, EPI_RELU>(65536, 512, 96, 0);
  fails += run<128, EPI_MASK>(65536, 256, 256, 0);
  printf(fails ? "GEMM_TEST FAIL\n" : "GEMM_TEST PASS\n");
  return fails;
}
