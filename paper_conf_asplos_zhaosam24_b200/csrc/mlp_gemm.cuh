// mlp_gemm.cuh — the cost-model MLP as tcgen05 tensor-core GEMMs over the candidate batch.
//
// Paper: the cost model C is the TenSet MLP, "4 linear layers and approximately 250K parameters"
// (PAPER.md L1056-1059); Felix back-propagates through it with PyTorch (L1053-1055) to get
// d O / d x (Algorithm 1 line 18, L917).  Only the INPUT gradient is needed — the weights are fixed
// during the search — so every layer is two GEMMs over the batch:
//     forward   Z_l     = H_{l-1} W_l^T + b_l,  H_l = relu(Z_l)
//     backward  delta_{l-1} = (delta_l W_l) (.) [Z_{l-1} > 0]
//
// One kernel template computes  D[M x N] = A[M x K] * B[N x K]^T  with both operands K-major fp16,
// split-precision: every fp32 operand x is carried as hi = fp16(x), lo = fp16(x - hi) and the
// product is accumulated as A_hi B_hi + A_hi B_lo + A_lo B_hi in fp32 TMEM (3 tcgen05.mma per K step;
// DESIGN.md "Precision").  Operand tiles arrive by TMA (SWIZZLE_128B) into a multi-stage mbarrier
// ring; one elected thread issues tcgen05.mma; all four warps drain TMEM (tcgen05.ld) in the
// epilogue, which fuses bias / ReLU / mask / head-GEMV / split-to-fp16 so no layer output is
// written in fp32 except the final d(loss)/d(phi).
#pragma once
#include <cstdint>
#include <cuda_fp16.h>
#include "sm100_ptx.cuh"

namespace felix {

enum EpiMode : int {
  EPI_RELU = 0,   // H = relu(acc + b)   -> out hi/lo, mask bits
  EPI_HEAD = 1,   // H = relu(acc + b);  c_part = H . w_L ;  delta = [Z>0] * (-w_L) -> out hi/lo
  EPI_MASK = 2,   // delta = acc (.) mask -> out hi/lo
  EPI_F32T = 3,   // out_f32[n][row] = acc  (n < n_valid), SoA for the DAG reverse kernel
};

struct GemmArgs {
  int M, N, K;
  const float* bias;          // [N]           RELU, HEAD
  const float* head_w;        // [N]           HEAD   (w_L, the last layer's single row)
  __half* out_hi;             // [M][ld_out]   RELU, HEAD, MASK
  __half* out_lo;
  int ld_out;
  uint32_t* mask_out;         // [N/32][ld_mask] RELU: bit i of word (w, row) = [z(row, 32w + i) > 0]
  const uint32_t* mask_in;    // [N/32][ld_mask] MASK
  int ld_mask;
  float* c_part;              // [N/BN][ld_c]  HEAD: per-N-tile partial of the head dot product
  int ld_c;
  float* out_f32;             // [n_valid][ld_f32]  F32T
  int ld_f32;
  int n_valid;
#ifdef FELIX_GEMM_TRACE
  unsigned long long* trace;  // [grid][8] globaltimer stamps (debug builds only)
#endif
};

#ifdef FELIX_GEMM_TRACE
__device__ __forceinline__ unsigned long long gtimer() { unsigned long long t; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t)); return t; }
#define GEMM_STAMP(slot) do { args.trace[(blockIdx.y * gridDim.x + blockIdx.x) * 8 + (slot)] = gtimer(); } while (0)
#else
#define GEMM_STAMP(slot) do {} while (0)
#endif

constexpr int GEMM_BM = 128;      // UMMA M (one CTA, cta_group::1)
constexpr int GEMM_BK = 64;       // fp16 elements per 128-byte swizzled row
constexpr int GEMM_UMMA_K = 16;   // K per tcgen05.mma kind::f16

template <int BN>
struct GemmCfg {
  static_assert(BN % 16 == 0 && BN >= 16 && BN <= 256, "UMMA N for M=128");
  static constexpr int A_BYTES = GEMM_BM * GEMM_BK * 2;             // one of hi / lo
  static constexpr int B_BYTES = BN * GEMM_BK * 2;
  static constexpr int B_BYTES_AL = (B_BYTES + 1023) / 1024 * 1024;  // keep every tile 1024-B aligned
  static constexpr int STAGE_BYTES = 2 * A_BYTES + 2 * B_BYTES_AL;
  static constexpr int MAX_STAGES = (200 * 1024) / STAGE_BYTES >= 4 ? 4 : (200 * 1024) / STAGE_BYTES;
  static constexpr int TX_BYTES = 2 * A_BYTES + 2 * B_BYTES;
  static constexpr int TMEM_COLS = BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : 256;
  // pipeline depth is chosen per launch (min(MAX_STAGES, K blocks)) so short-K GEMMs need less
  // shared memory and two CTAs can share an SM
  static constexpr int smem_bytes(int stages) { return 1024 /*align slack*/ + stages * STAGE_BYTES + 256 /*barriers*/; }
  static_assert(MAX_STAGES >= 2, "pipeline depth");
};

__device__ __forceinline__ void split_store16(__half* hi, __half* lo, const float (&v)[16]) {
  __align__(16) __half h[16];
  __align__(16) __half l[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) {
    h[i] = __float2half_rn(v[i]);
    l[i] = __float2half_rn(v[i] - __half2float(h[i]));
  }
  reinterpret_cast<uint4*>(hi)[0] = reinterpret_cast<const uint4*>(h)[0];
  reinterpret_cast<uint4*>(hi)[1] = reinterpret_cast<const uint4*>(h)[1];
  reinterpret_cast<uint4*>(lo)[0] = reinterpret_cast<const uint4*>(l)[0];
  reinterpret_cast<uint4*>(lo)[1] = reinterpret_cast<const uint4*>(l)[1];
}

template <int BN, int EPI>
__global__ void __launch_bounds__(128, 1)
mlp_gemm_kernel(const __grid_constant__ CUtensorMap tmA_hi, const __grid_constant__ CUtensorMap tmA_lo,
                const __grid_constant__ CUtensorMap tmB_hi, const __grid_constant__ CUtensorMap tmB_lo,
                const __grid_constant__ CUtensorMap tmC_hi, const __grid_constant__ CUtensorMap tmC_lo,
                GemmArgs args, int stages) {
  using Cfg = GemmCfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  // 1024-B alignment by offsetting the shared array itself (a round trip through uintptr_t would turn
  // every smem access into a generic LD/ST)
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full_bar  = reinterpret_cast<uint64_t*>(smem + stages * Cfg::STAGE_BYTES);
  uint64_t* empty_bar = full_bar + Cfg::MAX_STAGES;
  uint64_t* done_bar  = empty_bar + Cfg::MAX_STAGES;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(done_bar + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) GEMM_STAMP(0);
  const int m0 = blockIdx.x * GEMM_BM;
  const int n0 = blockIdx.y * BN;
  const int nkb = (args.K + GEMM_BK - 1) / GEMM_BK;

  auto a_hi = [&](int s) { return smem + s * Cfg::STAGE_BYTES; };
  auto a_lo = [&](int s) { return smem + s * Cfg::STAGE_BYTES + Cfg::A_BYTES; };
  auto b_hi = [&](int s) { return smem + s * Cfg::STAGE_BYTES + 2 * Cfg::A_BYTES; };
  auto b_lo = [&](int s) { return smem + s * Cfg::STAGE_BYTES + 2 * Cfg::A_BYTES + Cfg::B_BYTES_AL; };

  if (warp == 0 && lane == 0) {
    ptx::tma_prefetch_desc(&tmA_hi); ptx::tma_prefetch_desc(&tmA_lo);
    ptx::tma_prefetch_desc(&tmB_hi); ptx::tma_prefetch_desc(&tmB_lo);
    for (int s = 0; s < stages; ++s) { ptx::mbar_init(&full_bar[s], 1); ptx::mbar_init(&empty_bar[s], 1); }
    ptx::mbar_init(done_bar, 1);
    ptx::fence_barrier_init();
  }
  if (warp == 2) ptx::tmem_alloc(tmem_slot, Cfg::TMEM_COLS);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_d = *tmem_slot;
  // PDL: everything above overlapped the previous kernel's tail; operands are its outputs
  ptx::pdl_launch_dependents();
  ptx::pdl_wait();
  if (threadIdx.x == 0) GEMM_STAMP(1);

  if (warp == 0 && lane == 0) {
    // ---------------- TMA producer
    for (int kb = 0; kb < nkb; ++kb) {
      const int s = kb % stages;
      if (kb >= stages) ptx::mbar_wait(&empty_bar[s], ((kb / stages) - 1) & 1);
      ptx::mbar_arrive_expect_tx(&full_bar[s], Cfg::TX_BYTES);
      const int k0 = kb * GEMM_BK;
      ptx::tma_load_2d(a_hi(s), &tmA_hi, k0, m0, &full_bar[s]);
      ptx::tma_load_2d(a_lo(s), &tmA_lo, k0, m0, &full_bar[s]);
      ptx::tma_load_2d(b_hi(s), &tmB_hi, k0, n0, &full_bar[s]);
      ptx::tma_load_2d(b_lo(s), &tmB_lo, k0, n0, &full_bar[s]);
    }
  } else if (warp == 1 && lane == 0) {
    // ---------------- MMA issuer (single thread)
    constexpr uint32_t idesc = ptx::idesc_f16_f32(GEMM_BM, BN);
    for (int kb = 0; kb < nkb; ++kb) {
      const int s = kb % stages;
      ptx::mbar_wait(&full_bar[s], (kb / stages) & 1);
      if (kb == 0) GEMM_STAMP(2);
      ptx::tc_fence_after();
      const uint32_t ah = ptx::smem_u32(a_hi(s)), al = ptx::smem_u32(a_lo(s));
      const uint32_t bh = ptx::smem_u32(b_hi(s)), bl = ptx::smem_u32(b_lo(s));
#pragma unroll
      for (int kk = 0; kk < GEMM_BK / GEMM_UMMA_K; ++kk) {
        const uint32_t off = kk * GEMM_UMMA_K * 2;   // bytes along the 128-B swizzled row
        const uint32_t acc0 = (kb | kk) != 0;
        ptx::mma_f16_ss(tmem_d, ptx::sdesc_k_sw128(al + off), ptx::sdesc_k_sw128(bh + off), idesc, acc0);
        ptx::mma_f16_ss(tmem_d, ptx::sdesc_k_sw128(ah + off), ptx::sdesc_k_sw128(bl + off), idesc, 1u);
        ptx::mma_f16_ss(tmem_d, ptx::sdesc_k_sw128(ah + off), ptx::sdesc_k_sw128(bh + off), idesc, 1u);
      }
      ptx::mma_commit(&empty_bar[s]);   // frees this smem stage once the MMAs have read it
    }
    ptx::mma_commit(done_bar);          // accumulator complete
    GEMM_STAMP(3);
  }
  __syncwarp();

  // ---------------- epilogue: all 4 warps, warp w owns TMEM lanes [32w, 32w+32) = tile rows
  ptx::mbar_wait(done_bar, 0);
  if (threadIdx.x == 0) GEMM_STAMP(4);
  ptx::tc_fence_after();
  const int r_tile = warp * 32 + lane;              // row inside the 128-row tile
  const int row = m0 + r_tile;
  const bool row_ok = row < args.M;
  const uint32_t t_row = tmem_d + (static_cast<uint32_t>(warp * 32) << 16);
  float head_acc = 0.f;

  if constexpr (EPI == EPI_F32T) {
    // dL/dphi, transposed SoA [n][row]: consecutive lanes write consecutive rows (coalesced)
#pragma unroll 1
    for (int c = 0; c < BN; c += 32) {
      float v[32];
      {
        float a[16], b[16];
        ptx::tmem_ld16(t_row + c, a);
        ptx::tmem_ld16(t_row + c + 16, b);
#pragma unroll
        for (int i = 0; i < 16; ++i) { v[i] = a[i]; v[16 + i] = b[i]; }
      }
      const int n = n0 + c;
      if (row_ok) {
#pragma unroll
        for (int i = 0; i < 32; ++i)
          if (n + i < args.n_valid) args.out_f32[static_cast<size_t>(n + i) * args.ld_f32 + row] = v[i];
      }
    }
  } else {
    // hi/lo fp16 outputs: each 64-column chunk is written by the threads into a 128B-swizzled smem
    // tile (the TMA SWIZZLE_128B image: 16-B chunk q of row r lands at (q ^ (r & 7))), then stored
    // to global by one TMA bulk-tensor store per hi / lo — coalesced, ragged rows clipped by TMA.
#pragma unroll 1
    for (int c64 = 0; c64 < BN; c64 += 64) {
      const int chunk = c64 / 64;
      uint8_t* o_hi = a_hi(chunk & 1);
      uint8_t* o_lo = a_lo(chunk & 1);
      if (chunk >= 2) {
        if (threadIdx.x == 0) ptx::bulk_wait_read<1>();
        ptx::named_bar_sync(1, 128);
      }
#pragma unroll 1
      for (int c32 = 0; c32 < 64; c32 += 32) {
        const int c = c64 + c32;
        float v[32];
        {
          float a[16], b[16];
          ptx::tmem_ld16(t_row + c, a);
          ptx::tmem_ld16(t_row + c + 16, b);
#pragma unroll
          for (int i = 0; i < 16; ++i) { v[i] = a[i]; v[16 + i] = b[i]; }
        }
        const int n = n0 + c;
        if constexpr (EPI == EPI_RELU || EPI == EPI_HEAD) {
          uint32_t bits = 0;
#pragma unroll
          for (int i = 0; i < 32; ++i) {
            const float z = v[i] + __ldg(&args.bias[n + i]);
            const bool on = z > 0.f;
            bits |= (on ? 1u : 0u) << i;
            if constexpr (EPI == EPI_RELU) {
              v[i] = on ? z : 0.f;
            } else {
              const float w = __ldg(&args.head_w[n + i]);
              head_acc += (on ? z : 0.f) * w;
              v[i] = on ? -w : 0.f;          // delta_{L-1} = W_L^T (dL/dc = -1) (.) [Z > 0]
            }
          }
          if constexpr (EPI == EPI_RELU)
            if (row_ok) args.mask_out[static_cast<size_t>(n / 32) * args.ld_mask + row] = bits;
        } else {  // EPI_MASK
          const uint32_t bits = row_ok ? __ldg(&args.mask_in[static_cast<size_t>(n / 32) * args.ld_mask + row]) : 0u;
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = ((bits >> i) & 1u) ? v[i] : 0.f;
        }
        // split to fp16 hi / lo and write 4 x 16 B of this row into the swizzled tiles
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          uint32_t h[4], l[4];
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const float f0 = v[q * 8 + 2 * u], f1 = v[q * 8 + 2 * u + 1];
            const __half h0 = __float2half_rn(f0), h1 = __float2half_rn(f1);
            const __half l0 = __float2half_rn(f0 - __half2float(h0)), l1 = __float2half_rn(f1 - __half2float(h1));
            h[u] = static_cast<uint32_t>(__half_as_ushort(h0)) | (static_cast<uint32_t>(__half_as_ushort(h1)) << 16);
            l[u] = static_cast<uint32_t>(__half_as_ushort(l0)) | (static_cast<uint32_t>(__half_as_ushort(l1)) << 16);
          }
          const int q16 = c32 / 8 + q;                            // 16-B chunk index in the 128-B row
          const uint32_t off = r_tile * 128 + ((q16 ^ (r_tile & 7)) << 4);
          *reinterpret_cast<uint4*>(o_hi + off) = make_uint4(h[0], h[1], h[2], h[3]);
          *reinterpret_cast<uint4*>(o_lo + off) = make_uint4(l[0], l[1], l[2], l[3]);
        }
      }
      ptx::fence_proxy_async_smem();
      ptx::named_bar_sync(1, 128);
      if (threadIdx.x == 0) {
        ptx::tma_store_2d(&tmC_hi, n0 + c64, m0, o_hi);
        ptx::tma_store_2d(&tmC_lo, n0 + c64, m0, o_lo);
        ptx::bulk_commit();
      }
    }
    if (threadIdx.x == 0) ptx::bulk_wait<0>();
  }
  if constexpr (EPI == EPI_HEAD) {
    if (row_ok) args.c_part[static_cast<size_t>(blockIdx.y) * args.ld_c + row] = head_acc;
  }

  ptx::tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0) GEMM_STAMP(5);
  if (warp == 2) ptx::tmem_dealloc(tmem_d, Cfg::TMEM_COLS);
}

}  // namespace felix
