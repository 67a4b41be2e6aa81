// mlp_tile.cuh — tile-local fused MLP: one CTA (CG=1) or one 2-SM CTA pair (CG=2, tcgen05 cta_group::2)
// runs the whole forward + input-gradient backward of the TenSet cost model (dims [K0p, 512, 256, 256, 1],
// PAPER.md L1056-1059) for 128 (CG=1) or 256 (CG=2) candidates, with every activation kept on-chip.
//
// Why: the layer-by-layer chain (mlp_chain.cuh) pays, per layer, an L2 round trip of the activations
// (TMA store drain + TMA load latency), a grid-wide barrier and per-SM L2 bandwidth for re-read
// operands.  Here only the weights stream in (TMA ring); the A operand of every GEMM is written by the
// epilogue warps straight into shared memory in the UMMA 128-byte-swizzled K-major layout, and the
// accumulators live in TMEM.  Same math as the chain: split fp16 hi/lo, three tcgen05.mma per K step
// (A_lo B_hi + A_hi B_lo + A_hi B_hi), fp32 accumulation.
//
// CG=2 (default): a cluster of two CTAs on two SMs; MMAs are M=256 (128 rows per CTA, each CTA's A in
// its own smem) and every weight tile is split along N between the two CTAs, so each SM stages half
// of the weight bytes and the leader issues one instruction per 256 x N x 16 block (measured on B200:
// SS-mode tcgen05 at M=128 reads A+B from smem at 128 B/clk, so N<=128 single-SM MMAs are smem-bound
// and the per-SM weight ring is what limits the pipeline).
//
// Per tile (row r of the CTA's 128 rows = TMEM lane r; epilogue thread (quadrant q, half h) owns rows
// 32q..32q+31 and columns [64c + 32h, +32) of every 64-column chunk c of every layer, so the ReLU mask
// words it produces in the forward are exactly the ones it needs in the backward — kept in registers):
//   F1  Z1_c = phi W1[c]^T (4 chunks of 128, TMEM double buffer) -> H1 = relu(Z1 + b1) in 64-col chunks
//       Z2  += H1_j W2[:, j]^T                                     (TMEM 256 cols)
//   F2  H2_j = relu(Z2_j + b2) (smem)  ->  Z3 += H2_j W3[:, j]^T   (TMEM 256 cols)
//   F3  c = relu(Z3 + b3) . w4 (+ b4 in the reverse kernel);  m3 = [Z3 + b3 > 0]
//   B1  delta3_j = -w4 (.) m3 (smem)  ->  D2 += delta3_j W3^T[:, j]^T
//   B2  delta2_j = D2_j (.) m2 -> smem (all 4 chunks, 128 KB)
//   B3  D1_q = delta2 W2^T[q]^T (4 quarters of 128, TMEM double buffer) -> delta1 = D1_q (.) m1 (smem)
//       dphi += delta1_c W1^T[:, c]^T                              (TMEM 128 cols)
//   B4  dphi -> global, transposed [K0p][n] (the reverse DAG kernel's input)
// Warp roles (320 threads per CTA): warp 0 TMA producer, warp 1 MMA issuer (leader CTA only),
// warps 2..9 epilogue.
#pragma once
#include <cstdint>
#include <cuda_fp16.h>
#include "sm100_ptx.cuh"

namespace felix {

namespace tile {
constexpr int D1 = 512, D2 = 256, D3 = 256;   // TenSet hidden widths (this kernel's specialisation)
constexpr int THREADS = 320;
constexpr int EPI_WARPS = 8;
constexpr int CHUNK_BYTES = 2 * 128 * 64 * 2;            // hi + lo of one [128 x 64] A chunk
constexpr int HALF_BYTES = 128 * 64 * 2;
constexpr int RING_STAGE = 2 * 128 * 64 * 2;             // hi + lo of one <=128-row B tile
constexpr int RING = 2;
constexpr int R0_BYTES = 4 * CHUNK_BYTES;                // phi (2 chunks) + H buffers (2) | delta2 (4)
constexpr int SMEM_BYTES = 1024 + R0_BYTES + CHUNK_BYTES /*delta1*/ + RING * RING_STAGE + 512;
// TMEM columns
constexpr uint32_t T_Z1 = 0, T_Z3 = 0, T_D1 = 0;         // Z1: 2 x 128; Z3: 256; D1: 2 x 128
constexpr uint32_t T_Z2 = 256, T_D2 = 256, T_DPHI = 256; // Z2, D2: 256; dphi: 128
}  // namespace tile

struct TileParams {
  CUtensorMap phi_hi, phi_lo;          // [n][K0p]   box 128 x 64
  CUtensorMap w1_hi, w1_lo;            // [512][K0p] box 128/CG x 64
  CUtensorMap w2_hi, w2_lo;            // [256][512] box 128 x 64
  CUtensorMap w3_hi, w3_lo;            // [256][256] box 128 x 64
  CUtensorMap w3t_hi, w3t_lo;          // [256][256] box 128 x 64 (W3^T)
  CUtensorMap w2t_hi, w2t_lo;          // [512][256] box 128/CG x 64 (W2^T)
  CUtensorMap w1t_hi, w1t_lo;          // [K0p][512] box K0p/CG x 64 (W1^T)
  const float* b1;
  const float* b2;
  const float* b3;
  const float* w4;
  float* c_part;                       // [2][ld] head partials (one per column half)
  float* dphi;                         // [K0p][ld]
  CUtensorMap dphi_map;                // fp32 [K0p][ld], box {128 rows, K0p}: B4 as one TMA store per tile
  int dphi_tma;                        // 1: B4 staged in shared memory + TMA store; 0: per-thread stores
  int ld;
  int n;                               // rows (candidates)
  int n_tiles;                         // 128-row tiles
  int k0p;                             // padded feature count (<= 128, multiple of 32)
  int n_valid;                         // real feature count
  int d2_exact;                        // B1 takes the exact 0/1 mask [Z3 > 0] (w3t = W3^T diag(-w4)): 2 passes
  uint32_t idesc_128, idesc_256, idesc_k0p;   // M = 128*CG; N = 128 / 256 / K0p
  unsigned long long* trace;           // FELIX_TILE_TRACE builds only: [grid][32] timestamps
};

#ifdef FELIX_TILE_TRACE
#define TILE_STAMP(slot) do { if (t == 0) { unsigned long long g_; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g_)); \
    P.trace[blockIdx.x * 32 + (slot)] = g_; } } while (0)
#else
#define TILE_STAMP(slot) do {} while (0)
#endif

namespace tile {

template <int CG>
__device__ __forceinline__ void mma(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  if constexpr (CG == 2) ptx::mma_f16_ss_cg2(d, a, b, idesc, acc);
  else ptx::mma_f16_ss(d, a, b, idesc, acc);
}
template <int CG>
__device__ __forceinline__ void commit(uint64_t* bar) {
  if constexpr (CG == 2) ptx::mma_commit_mc(bar, 0x3);
  else ptx::mma_commit(bar);
}
// barriers that receive arrivals from the peer CTA are waited on with cluster-scope acquire
template <int CG>
__device__ __forceinline__ void wait_k(uint64_t* bar, uint32_t k) {
  if constexpr (CG == 2) ptx::mbar_wait_cluster(bar, k & 1u);
  else ptx::mbar_wait(bar, k & 1u);
}
// arrive on the LEADER CTA's copy of `bar` (this CTA's own for CG=1)
template <int CG>
__device__ __forceinline__ void arrive_leader(uint64_t* bar) {
  if constexpr (CG == 2) ptx::mbar_arrive_cluster(ptx::mapa_shared(ptx::smem_u32(bar), 0));
  else ptx::mbar_arrive(bar);
}

// 4 K-steps x 3 split passes of one 64-wide K block: D (+)= A[128 x 64] * B[N x 64]^T
template <int CG>
__device__ __forceinline__ void mma_kblock(uint32_t d, uint32_t a_hi, uint32_t a_lo, uint32_t b_hi, uint32_t b_lo,
                                           uint32_t idesc, bool accumulate, bool a_exact = false) {
  const uint64_t dah = ptx::sdesc_k_sw128(a_hi), dal = ptx::sdesc_k_sw128(a_lo);
  const uint64_t dbh = ptx::sdesc_k_sw128(b_hi), dbl = ptx::sdesc_k_sw128(b_lo);
#pragma unroll
  for (int kk = 0; kk < 4; ++kk) {           // +32 B along K = +2 in the descriptor's address field
    if (!a_exact) mma<CG>(d, dal + 2 * kk, dbh + 2 * kk, idesc, (accumulate || kk) ? 1u : 0u);   // A lo = 0 if exact
    mma<CG>(d, dah + 2 * kk, dbl + 2 * kk, idesc, (!a_exact || accumulate || kk) ? 1u : 0u);
    mma<CG>(d, dah + 2 * kk, dbh + 2 * kk, idesc, 1u);
  }
}

// one thread's 32 values of a row -> fp16 hi/lo, written into a swizzled [128 x 64] chunk (column
// half h = this thread's 32 columns = 16-byte chunks 4h..4h+3 of the 128-byte row)
__device__ __forceinline__ void store_split32(uint8_t* chunk_hi, uint8_t* chunk_lo, int r, int h, const float (&v)[32]) {
#pragma unroll
  for (int qq = 0; qq < 4; ++qq) {
    uint32_t hw[4], lw[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const float2 f = make_float2(v[qq * 8 + 2 * u], v[qq * 8 + 2 * u + 1]);
      const __half2 hh = __float22half2_rn(f);
      const float2 back = __half22float2(hh);
      const __half2 ll = __float22half2_rn(make_float2(f.x - back.x, f.y - back.y));
      hw[u] = *reinterpret_cast<const uint32_t*>(&hh);
      lw[u] = *reinterpret_cast<const uint32_t*>(&ll);
    }
    const int q16 = h * 4 + qq;
    const uint32_t off = r * 128 + ((q16 ^ (r & 7)) << 4);
    *reinterpret_cast<uint4*>(chunk_hi + off) = make_uint4(hw[0], hw[1], hw[2], hw[3]);
    *reinterpret_cast<uint4*>(chunk_lo + off) = make_uint4(lw[0], lw[1], lw[2], lw[3]);
  }
}

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, float (&v)[32]) {
  uint32_t x[32];
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 "
               "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
               "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
               : "=r"(x[0]), "=r"(x[1]), "=r"(x[2]), "=r"(x[3]), "=r"(x[4]), "=r"(x[5]), "=r"(x[6]), "=r"(x[7]),
                 "=r"(x[8]), "=r"(x[9]), "=r"(x[10]), "=r"(x[11]), "=r"(x[12]), "=r"(x[13]), "=r"(x[14]), "=r"(x[15]),
                 "=r"(x[16]), "=r"(x[17]), "=r"(x[18]), "=r"(x[19]), "=r"(x[20]), "=r"(x[21]), "=r"(x[22]), "=r"(x[23]),
                 "=r"(x[24]), "=r"(x[25]), "=r"(x[26]), "=r"(x[27]), "=r"(x[28]), "=r"(x[29]), "=r"(x[30]), "=r"(x[31])
               : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(x[i]);
}

// epilogue-side "done with smem writes / TMEM reads" arrivals (one per warp, on the leader's barrier)
template <int CG>
__device__ __forceinline__ void warp_arrive_smem(uint64_t* bar, int lane) {
  ptx::fence_proxy_async_smem();   // generic-proxy smem writes -> visible to the tensor core (async proxy)
  __syncwarp();
  if (lane == 0) arrive_leader<CG>(bar);
}
template <int CG>
__device__ __forceinline__ void warp_arrive_tmem(uint64_t* bar, int lane) {
  ptx::tc_fence_before();
  __syncwarp();
  if (lane == 0) arrive_leader<CG>(bar);
}

// epilogue: write the next H / delta3 chunk into the H buffer of use `hseq` (after the MMA freed it)
template <int CG>
__device__ __forceinline__ void put_h(uint8_t* R0, uint64_t* a_free, uint64_t* a_ready, uint32_t& hseq, int r, int h,
                                      int lane, const float (&v)[32]) {
  const int b = hseq & 1;
  uint8_t* buf = R0 + (2 + b) * CHUNK_BYTES;
  if (hseq >= 2) wait_k<1>(&a_free[b], (hseq >> 1) - 1);
  store_split32(buf, buf + HALF_BYTES, r, h, v);
  warp_arrive_smem<CG>(&a_ready[b], lane);
  ++hseq;
}

}  // namespace tile

template <int CG>
__global__ void __launch_bounds__(tile::THREADS, 1) mlp_tile_kernel(const __grid_constant__ TileParams P) {
  using namespace tile;
  extern __shared__ uint8_t smem_raw[];
  // 1024-B alignment by offsetting the shared array itself (a round trip through uintptr_t would turn
  // every smem access into a generic LD/ST)
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* R0 = smem;                                  // 4 chunks: phi0 phi1 H0 H1 | delta2_0..3
  uint8_t* RD1 = R0 + R0_BYTES;                        // delta1 chunk
  uint8_t* RING_BASE = RD1 + CHUNK_BYTES;
  uint64_t* bars = reinterpret_cast<uint64_t*>(RING_BASE + RING * RING_STAGE);
  uint64_t* ring_full = bars + 0;    // [2]   (leader: producer arms, both CTAs' TMA complete)
  uint64_t* ring_empty = bars + 2;   // [2]   (both: MMA commit)
  uint64_t* phi_full = bars + 4;     //       (leader)
  uint64_t* phi_free = bars + 5;     //       (both: MMA commit)
  uint64_t* a_ready = bars + 6;      // [3]   (leader: epilogue warps of both CTAs) H0, H1, delta1
  uint64_t* a_free = bars + 9;       // [3]   (both: MMA commit)
  uint64_t* z1_full = bars + 12;     // [2]   (both)
  uint64_t* z1_free = bars + 14;     // [2]   (leader)
  uint64_t* z2_full = bars + 16;
  uint64_t* z3_full = bars + 17;
  uint64_t* d2_full = bars + 18;
  uint64_t* d2_ready = bars + 19;    //       (leader) delta2 chunks written
  uint64_t* d1_full = bars + 20;     // [2]
  uint64_t* d1_free = bars + 22;     // [2]   (leader)
  uint64_t* dphi_full = bars + 24;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 26);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = (CG == 2) ? ptx::cluster_ctarank() : 0u;
  auto phi_c = [&](int kc) { return R0 + kc * CHUNK_BYTES; };
  auto hbuf = [&](int b) { return R0 + (2 + b) * CHUNK_BYTES; };
  auto d2c = [&](int j) { return R0 + j * CHUNK_BYTES; };
  auto ring_hi = [&](int s) { return RING_BASE + s * RING_STAGE; };

  if (warp == 0 && lane == 0) {
    const uint32_t epi_arrivals = EPI_WARPS * CG;
    for (int s = 0; s < RING; ++s) { ptx::mbar_init(&ring_full[s], 1); ptx::mbar_init(&ring_empty[s], 1); }
    ptx::mbar_init(phi_full, 1);
    ptx::mbar_init(phi_free, 1);
    for (int b = 0; b < 3; ++b) { ptx::mbar_init(&a_ready[b], epi_arrivals); ptx::mbar_init(&a_free[b], 1); }
    for (int b = 0; b < 2; ++b) {
      ptx::mbar_init(&z1_full[b], 1); ptx::mbar_init(&z1_free[b], epi_arrivals);
      ptx::mbar_init(&d1_full[b], 1); ptx::mbar_init(&d1_free[b], epi_arrivals);
    }
    ptx::mbar_init(z2_full, 1);
    ptx::mbar_init(z3_full, 1);
    ptx::mbar_init(d2_full, 1);
    ptx::mbar_init(d2_ready, epi_arrivals);
    ptx::mbar_init(dphi_full, 1);
    ptx::fence_barrier_init();
  }
  if (warp == 1) {
    if constexpr (CG == 2) ptx::tmem_alloc_cg2(tmem_slot, 512);
    else ptx::tmem_alloc(tmem_slot, 512);
  }
  ptx::tc_fence_before();
  if constexpr (CG == 2) ptx::cluster_sync();
  else __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  ptx::pdl_launch_dependents();
  ptx::pdl_wait();                                    // phi comes from the forward DAG kernel

  const int n_units = (P.n_tiles + CG - 1) / CG;      // 128*CG-row units
  const int G = gridDim.x / CG;
  const int unit0 = blockIdx.x / CG;
  const int n_my = unit0 < n_units ? (n_units - unit0 + G - 1) / G : 0;

  if (warp == 0) {
    if (lane == 0) {
      // ================================================================ TMA producer (both CTAs)
      uint32_t it = 0;                                // ring entries issued
      const uint32_t full_leader0 = (CG == 2) ? ptx::mapa_shared(ptx::smem_u32(&ring_full[0]), 0) : 0u;
      const uint32_t phi_leader = (CG == 2) ? ptx::mapa_shared(ptx::smem_u32(phi_full), 0) : 0u;
      auto tma = [&](void* dst, const CUtensorMap* m, int c0, int c1, uint64_t* bar_local, uint32_t bar_leader) {
        if constexpr (CG == 2) ptx::tma_load_2d_cg2(dst, m, c0, c1, bar_leader);
        else ptx::tma_load_2d(dst, m, c0, c1, bar_local);
        (void)bar_local; (void)bar_leader;
      };
      // one ring entry: rows [row0 + rank*rows, +rows) x 64 K columns at k0, hi and lo
      auto load_b = [&](const CUtensorMap* mh, const CUtensorMap* ml, int rows, int k0, int row0) {
        const int s = it % RING;
        if (it >= RING) wait_k<1>(&ring_empty[s], it / RING - 1);
        if (rank == 0) ptx::mbar_arrive_expect_tx(&ring_full[s], static_cast<uint32_t>(rows) * 64 * 2 * 2 * CG);
        const uint32_t bl = full_leader0 + s * 8;
        tma(ring_hi(s), mh, k0, row0 + static_cast<int>(rank) * rows, &ring_full[s], bl);
        tma(ring_hi(s) + HALF_BYTES, ml, k0, row0 + static_cast<int>(rank) * rows, &ring_full[s], bl);
        ++it;
      };
      // logical GEMM step of width N: sub-entries of <= 128 rows per CTA
      auto load_n = [&](const CUtensorMap* mh, const CUtensorMap* ml, int N, int k0, int n0) {
        const int per = N / CG;
        if (per <= 128) load_b(mh, ml, per, k0, n0);
        else for (int s = 0; s < per / 128; ++s) load_b(mh, ml, 128, k0, n0 + s * 128 * CG);
      };
      for (int t = 0; t < n_my; ++t) {
        const int unit = unit0 + t * G;
        const int m0 = (unit * CG + static_cast<int>(rank)) * 128;
        TILE_STAMP(16);
        if (t > 0) wait_k<1>(phi_free, t - 1);
        if (rank == 0) ptx::mbar_arrive_expect_tx(phi_full, 2 * CHUNK_BYTES * CG);
        for (int kc = 0; kc < 2; ++kc) {
          tma(phi_c(kc), &P.phi_hi, kc * 64, m0, phi_full, phi_leader);
          tma(phi_c(kc) + HALF_BYTES, &P.phi_lo, kc * 64, m0, phi_full, phi_leader);
        }
        // F1: Z1_c (two K blocks), then Z2 += H1 of the previous chunk (two 64-col K blocks)
        for (int c = 0; c <= D1 / 128; ++c) {
          if (c < D1 / 128)
            for (int kc = 0; kc < 2; ++kc) load_n(&P.w1_hi, &P.w1_lo, 128, kc * 64, c * 128);
          if (c >= 1)
            for (int s = 0; s < 2; ++s) load_n(&P.w2_hi, &P.w2_lo, D2, ((c - 1) * 2 + s) * 64, 0);
        }
        for (int j = 0; j < D2 / 64; ++j) load_n(&P.w3_hi, &P.w3_lo, D3, j * 64, 0);      // F2
        for (int j = 0; j < D3 / 64; ++j) load_n(&P.w3t_hi, &P.w3t_lo, D2, j * 64, 0);    // B1
        auto d1q = [&](int q) { for (int kc = 0; kc < D2 / 64; ++kc) load_n(&P.w2t_hi, &P.w2t_lo, 128, kc * 64, q * 128); };
        auto dph = [&](int c) { load_n(&P.w1t_hi, &P.w1t_lo, P.k0p, c * 64, 0); };
        d1q(0); d1q(1); dph(0); dph(1); d1q(2); dph(2); dph(3); d1q(3); dph(4); dph(5); dph(6); dph(7);
        TILE_STAMP(18);
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && rank == 0) {
      // ================================================================ MMA issuer (leader CTA)
      uint32_t it = 0;                                // ring entries consumed
      uint32_t hseq = 0, d1seq = 0, z1seq = 0, d1accseq = 0;
      // one logical GEMM step of width N into accumulator d (A = one 64-wide K block in smem)
      auto step = [&](uint32_t d, uint8_t* a_chunk, int N, uint32_t idesc, bool accumulate, bool a_exact = false) {
        const int per = N / CG;
        const int nsub = per <= 128 ? 1 : per / 128;
        const uint32_t ah = ptx::smem_u32(a_chunk), al = ah + HALF_BYTES;
        for (int s = 0; s < nsub; ++s) {
          const int slot = it % RING;
          wait_k<CG>(&ring_full[slot], it / RING);
          ptx::tc_fence_after();
          const uint32_t bh = ptx::smem_u32(ring_hi(slot));
          mma_kblock<CG>(d + s * (N / nsub), ah, al, bh, bh + HALF_BYTES, idesc, accumulate, a_exact);
          commit<CG>(&ring_empty[slot]);
          ++it;
        }
      };
      // MMA instruction descriptor of a logical N=256 step (two N=128 sub-MMAs when CG=1)
      const uint32_t id_n256 = (CG == 2) ? P.idesc_256 : P.idesc_128;
      for (int t = 0; t < n_my; ++t) {
        TILE_STAMP(0);
        wait_k<CG>(phi_full, t);
        TILE_STAMP(1);
        ptx::tc_fence_after();
        auto consume_h = [&](uint32_t dacc, int N, uint32_t idesc, bool accumulate, bool a_exact = false) {
          const int b = hseq & 1;
          wait_k<CG>(&a_ready[b], hseq >> 1);
          ptx::tc_fence_after();
          step(dacc, hbuf(b), N, idesc, accumulate, a_exact);
          commit<CG>(&a_free[b]);
          ++hseq;
        };
        // ---- F1
        for (int c = 0; c <= D1 / 128; ++c) {
          if (c < D1 / 128) {
            const int b = z1seq & 1;
            if (z1seq >= 2) wait_k<CG>(&z1_free[b], (z1seq >> 1) - 1);
            ptx::tc_fence_after();
            for (int kc = 0; kc < 2; ++kc) step(tmem + T_Z1 + b * 128, phi_c(kc), 128, P.idesc_128, kc > 0);
            commit<CG>(&z1_full[b]);
            ++z1seq;
          }
          if (c >= 1)
            for (int s = 0; s < 2; ++s) consume_h(tmem + T_Z2, D2, id_n256, c > 1 || s > 0);
        }
        TILE_STAMP(2);
        commit<CG>(z2_full);
        // ---- F2: Z3 += H2_j
        for (int j = 0; j < D2 / 64; ++j) consume_h(tmem + T_Z3, D3, id_n256, j > 0);
        TILE_STAMP(3);
        commit<CG>(z3_full);
        // ---- B1: D2 += delta3_j W3^T
        for (int j = 0; j < D3 / 64; ++j) consume_h(tmem + T_D2, D2, id_n256, j > 0, P.d2_exact != 0);
        TILE_STAMP(4);
        commit<CG>(d2_full);
        // ---- B3
        wait_k<CG>(d2_ready, t);
        TILE_STAMP(5);
        ptx::tc_fence_after();
        auto d1q = [&](int q) {
          const int b = d1accseq & 1;
          if (d1accseq >= 2) wait_k<CG>(&d1_free[b], (d1accseq >> 1) - 1);
          ptx::tc_fence_after();
          for (int kc = 0; kc < D2 / 64; ++kc) step(tmem + T_D1 + b * 128, d2c(kc), 128, P.idesc_128, kc > 0);
          commit<CG>(&d1_full[b]);
          ++d1accseq;
          // R0 (phi | delta2) is last read by D1_3: the next tile's phi load may overwrite it after this
          if (q == 3) commit<CG>(phi_free);
        };
        auto dph = [&](int c) {
          wait_k<CG>(&a_ready[2], d1seq);
          ptx::tc_fence_after();
          step(tmem + T_DPHI, RD1, P.k0p, P.idesc_k0p, c > 0);
          commit<CG>(&a_free[2]);
          ++d1seq;
        };
        d1q(0); d1q(1); dph(0); dph(1); d1q(2); dph(2); dph(3); d1q(3); dph(4); dph(5); dph(6); dph(7);
        TILE_STAMP(6);
        commit<CG>(dphi_full);
      }
    }
  } else {
    // ================================================================ epilogue warps 2..9 (both CTAs)
    const int q = warp & 3;                 // TMEM lane quadrant
    const int h = (warp - 2) >> 2;          // column half of every 64-column chunk
    const int r = q * 32 + lane;            // tile row
    const uint32_t lane_base = static_cast<uint32_t>(q * 32) << 16;
    uint32_t hseq = 0, d1seq = 0, z1seq = 0, d1accseq = 0;
    for (int t = 0; t < n_my; ++t) {
      const int unit = unit0 + t * G;
      const int m0 = (unit * CG + static_cast<int>(rank)) * 128;
      const int row = m0 + r;
      const bool row_ok = row < P.n;
      if (t > 0 && P.dphi_tma) {
        // the previous tile's dL/dphi store has read its staging (the H buffers written again below)
        if (warp == 2 && lane == 0) ptx::bulk_wait_read<0>();
        ptx::named_bar_sync(1, EPI_WARPS * 32);
      }
      uint32_t m1w[D1 / 64], m2w[D2 / 64], m3w[D3 / 64];
      float head = 0.f;
      // ---- F1: drain Z1_c (128 columns) -> H1 chunks 2c, 2c+1
      for (int c = 0; c < D1 / 128; ++c) {
        const int b = z1seq & 1;
        wait_k<1>(&z1_full[b], z1seq >> 1);
        if (warp == 2 && lane == 0 && c == 0) TILE_STAMP(8);
        ptx::tc_fence_after();
        for (int s = 0; s < 2; ++s) {
          float v[32];
          tile::tmem_ld32(tmem + lane_base + T_Z1 + b * 128 + s * 64 + h * 32, v);
          if (s == 1) warp_arrive_tmem<CG>(&z1_free[b], lane);
          const int n0 = c * 128 + s * 64 + h * 32;
          uint32_t bits = 0;
#pragma unroll
          for (int i = 0; i < 32; ++i) {
            const float z = v[i] + __ldg(&P.b1[n0 + i]);
            const bool on = z > 0.f;
            bits |= (on ? 1u : 0u) << i;
            v[i] = on ? z : 0.f;
          }
          m1w[2 * c + s] = bits;
          tile::put_h<CG>(R0, a_free, a_ready, hseq, r, h, lane, v);
        }
        ++z1seq;
      }
      if (warp == 2 && lane == 0) TILE_STAMP(9);
      // ---- F2: drain Z2_j -> H2_j
      wait_k<1>(z2_full, t);
      if (warp == 2 && lane == 0) TILE_STAMP(10);
      ptx::tc_fence_after();
      for (int j = 0; j < D2 / 64; ++j) {
        float v[32];
        tile::tmem_ld32(tmem + lane_base + T_Z2 + j * 64 + h * 32, v);
        const int n0 = j * 64 + h * 32;
        uint32_t bits = 0;
#pragma unroll
        for (int i = 0; i < 32; ++i) {
          const float z = v[i] + __ldg(&P.b2[n0 + i]);
          const bool on = z > 0.f;
          bits |= (on ? 1u : 0u) << i;
          v[i] = on ? z : 0.f;
        }
        m2w[j] = bits;
        tile::put_h<CG>(R0, a_free, a_ready, hseq, r, h, lane, v);
      }
      if (warp == 2 && lane == 0) TILE_STAMP(11);
      // ---- F3: drain Z3 -> head partial, m3
      wait_k<1>(z3_full, t);
      if (warp == 2 && lane == 0) TILE_STAMP(12);
      ptx::tc_fence_after();
      for (int j = 0; j < D3 / 64; ++j) {
        float v[32];
        tile::tmem_ld32(tmem + lane_base + T_Z3 + j * 64 + h * 32, v);
        const int n0 = j * 64 + h * 32;
        uint32_t bits = 0;
#pragma unroll
        for (int i = 0; i < 32; ++i) {
          const float z = v[i] + __ldg(&P.b3[n0 + i]);
          const bool on = z > 0.f;
          bits |= (on ? 1u : 0u) << i;
          head += (on ? z : 0.f) * __ldg(&P.w4[n0 + i]);
        }
        m3w[j] = bits;
      }
      if (row_ok) P.c_part[static_cast<size_t>(h) * P.ld + row] = head;
      if (warp == 2 && lane == 0) TILE_STAMP(13);
      // ---- B1: delta3_j = -w4 (.) m3
      for (int j = 0; j < D3 / 64; ++j) {
        float v[32];
        const int n0 = j * 64 + h * 32;
#pragma unroll
        for (int i = 0; i < 32; ++i) v[i] = ((m3w[j] >> i) & 1u) ? (P.d2_exact ? 1.f : -__ldg(&P.w4[n0 + i])) : 0.f;
        tile::put_h<CG>(R0, a_free, a_ready, hseq, r, h, lane, v);
      }
      if (warp == 2 && lane == 0) TILE_STAMP(14);
      // ---- B2: drain D2 (.) m2 -> delta2 chunks (all four, 128 KB)
      wait_k<1>(d2_full, t);
      if (warp == 2 && lane == 0) TILE_STAMP(15);
      ptx::tc_fence_after();
      for (int j = 0; j < D2 / 64; ++j) {
        float v[32];
        tile::tmem_ld32(tmem + lane_base + T_D2 + j * 64 + h * 32, v);
#pragma unroll
        for (int i = 0; i < 32; ++i) v[i] = ((m2w[j] >> i) & 1u) ? v[i] : 0.f;
        tile::store_split32(d2c(j), d2c(j) + HALF_BYTES, r, h, v);
      }
      ptx::tc_fence_before();
      tile::warp_arrive_smem<CG>(d2_ready, lane);
      if (warp == 2 && lane == 0) TILE_STAMP(24);
      // ---- B3: drain D1_q (.) m1 -> delta1 chunks (two per quarter)
      for (int qq = 0; qq < D1 / 128; ++qq) {
        const int b = d1accseq & 1;
        wait_k<1>(&d1_full[b], d1accseq >> 1);
        ptx::tc_fence_after();
        for (int s = 0; s < 2; ++s) {
          const int c = qq * 2 + s;                   // delta1 chunk (64 columns)
          float v[32];
          tile::tmem_ld32(tmem + lane_base + T_D1 + b * 128 + s * 64 + h * 32, v);
          if (s == 1) warp_arrive_tmem<CG>(&d1_free[b], lane);
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = ((m1w[c] >> i) & 1u) ? v[i] : 0.f;
          if (d1seq >= 1) wait_k<1>(&a_free[2], d1seq - 1);
          tile::store_split32(RD1, RD1 + HALF_BYTES, r, h, v);
          tile::warp_arrive_smem<CG>(&a_ready[2], lane);
          ++d1seq;
        }
        ++d1accseq;
      }
      if (warp == 2 && lane == 0) TILE_STAMP(25);
      // ---- B4: dphi -> global [k][row]
      wait_k<1>(dphi_full, t);
      if (warp == 2 && lane == 0) TILE_STAMP(26);
      ptx::tc_fence_after();
      if (P.dphi_tma) {
        // staged [K0p][128 rows] fp32 in the H buffers (free here: every MMA reading them has completed
        // before dphi_full) and written by one TMA store (per-thread fp32 stores took ~2.4 us per tile)
        float* stg = reinterpret_cast<float*>(R0 + 2 * CHUNK_BYTES);
        for (int c = h * 32; c < P.k0p; c += 64) {
          float v[32];
          tile::tmem_ld32(tmem + lane_base + T_DPHI + c, v);
#pragma unroll
          for (int i = 0; i < 32; ++i)
            if (c + i < P.k0p) stg[(c + i) * 128 + r] = v[i];
        }
        ptx::tc_fence_before();
        ptx::fence_proxy_async_smem();
        ptx::named_bar_sync(1, EPI_WARPS * 32);
        if (warp == 2 && lane == 0) {
          asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
                       :: "l"(reinterpret_cast<uint64_t>(&P.dphi_map)), "r"(m0), "r"(0), "r"(ptx::smem_u32(stg)) : "memory");
          ptx::bulk_commit();
        }
      } else {
        for (int c = h * 32; c < P.k0p; c += 64) {
          float v[32];
          tile::tmem_ld32(tmem + lane_base + T_DPHI + c, v);
          if (row_ok) {
#pragma unroll
            for (int i = 0; i < 32; ++i)
              if (c + i < P.n_valid) P.dphi[static_cast<size_t>(c + i) * P.ld + row] = v[i];
          }
        }
        ptx::tc_fence_before();
      }
      if (warp == 2 && lane == 0) TILE_STAMP(27);
    }
    if (warp == 2 && lane == 0) ptx::bulk_wait<0>();   // the last dL/dphi store complete before exit
  }
  ptx::tc_fence_before();
  if constexpr (CG == 2) ptx::cluster_sync();
  else __syncthreads();
  if (warp == 1) {
    if constexpr (CG == 2) ptx::tmem_dealloc_cg2(tmem, 512);
    else ptx::tmem_dealloc(tmem, 512);
  }
}

}  // namespace felix
