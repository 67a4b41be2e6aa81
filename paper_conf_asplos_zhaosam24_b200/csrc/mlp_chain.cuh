// mlp_chain.cuh — the whole cost-model MLP of one Adam step (forward + input-gradient backward,
// 2(L-1) GEMM layers) in ONE persistent kernel.
//
// Why: at the C2 population (4096 candidates) every layer is a few microseconds of tensor work, and
// separate launches cost ~4 us each at the kernel boundary (launch ramp, prologue, drain) even
// with PDL + CUDA graphs.  Here one CTA per SM loops over the tiles of every layer; layers are
// separated by a grid-wide release/acquire barrier.  Per layer the math is the one of
// mlp_gemm.cuh (split fp16 hi/lo, 3 tcgen05.mma per
// K step, fp32 TMEM accumulation) and the epilogues are the same (bias/ReLU/mask, head GEMV,
// -w_L seed, dL/dphi transpose).
//
// Warp roles (320 threads): warp 0 = TMA producer, warp 1 = MMA issuer (one elected thread),
// warps 2..9 = epilogue: warp w drains TMEM lanes 32*(w%4)..+31, warps w and w+4 split every
// 64-column chunk into two 32-column halves (two warps per SM sub-partition hide the latency of
// the convert/split chains).  TMEM holds two 128-column accumulators so the epilogue of tile i
// overlaps the MMAs of tile i+1.
//
// CG = 2 (2-SM pairs, tcgen05 cta_group::2): a cluster of two CTAs computes 256-row x bn tiles (rows
// 256p + 128 rank ...); each CTA loads its own 128 A rows and HALF of the tile's weight rows (B split
// along N), the leader issues M=256 MMAs that read A and B from both CTAs' shared memory, and each
// CTA's TMEM receives the 128 x bn accumulator of its own rows.  Per SM the weight bytes of a tile
// halve (C2: 1376 -> 1128 KB ingested per Adam step); every epilogue, flag and own-chunk reuse stays
// per CTA (its own 128-row block), exactly as with CG = 1.  TMA loads of both CTAs complete on the
// leader's full barrier (armed by the leader with both CTAs' bytes); MMA commits are multicast to both
// CTAs' empty / accumulator-ready barriers; the epilogues of both CTAs arrive on the leader's
// accumulator-drained and own-chunk barriers.
#pragma once
#include <cstdint>
#include <cuda_fp16.h>
#include "sm100_ptx.cuh"
#include "mlp_gemm.cuh"

namespace felix {

constexpr int CHAIN_MAX_LAYERS = 14;
constexpr int CHAIN_BN_MAX = 128;
#ifndef FELIX_CHAIN_STAGES
#define FELIX_CHAIN_STAGES 2
#endif
constexpr int CHAIN_STAGES = FELIX_CHAIN_STAGES;
constexpr int CHAIN_EPI_BUFS = CHAIN_STAGES >= 3 ? 1 : 2;   // epilogue staging buffers (double-buffered when smem allows)
// Epilogue warps: 8 = two warps per TMEM lane quadrant, each draining a 32-column half of every 64-column
// chunk (16 = four warps, 16-column slices).  Measured at C2 (tools/microbench/chain_trace.cu): 16 warps are
// no faster (37.3 vs 37.4 us per chain): the chunk epilogue is bound by the SM sub-partitions' issue slots
// (~8 instructions per element), not by per-warp latency.
#ifndef FELIX_CHAIN_EPI_WARPS
#define FELIX_CHAIN_EPI_WARPS 8
#endif
// NCAT = 1: the B tile of a stage is [B_hi ; B_lo] (2bn rows, contiguous), and the split product takes
// two MMAs per K step instead of three: A_hi x [B_hi ; B_lo] (N = 2bn, accumulator columns [0, 2bn)) and
// A_lo x B_hi (N = bn, accumulated into [0, bn)); the epilogue adds the two halves.  Shared-memory
// operand reads per K step fall from 3(128 + bn) to (128 + 2bn) + (128 + bn) rows: the mainloop is bound
// by the SM's shared-memory port (TMA writes + MMA operand reads), measured in tools/microbench/tma_ingest.cu.
#ifndef FELIX_CHAIN_NCAT
#define FELIX_CHAIN_NCAT 1
#endif
constexpr int CHAIN_EPI_WARPS = FELIX_CHAIN_EPI_WARPS;
constexpr int CHAIN_THREADS = 64 + 32 * CHAIN_EPI_WARPS;
constexpr int CHAIN_EPI_NQ = CHAIN_EPI_WARPS / 4;            // epilogue warps per TMEM lane quadrant
constexpr int CHAIN_EPI_CPW = 64 / CHAIN_EPI_NQ;             // columns of each 64-column chunk per warp (16 or 32)
static_assert(CHAIN_EPI_CPW == 16 || CHAIN_EPI_CPW == 32, "8 or 16 epilogue warps");
constexpr int CHAIN_A_BYTES = GEMM_BM * GEMM_BK * 2;                 // 16 KB (one of hi / lo)
#ifndef FELIX_CHAIN_STAGE_BN
#define FELIX_CHAIN_STAGE_BN CHAIN_BN_MAX
#endif
constexpr int CHAIN_B_BYTES = FELIX_CHAIN_STAGE_BN * GEMM_BK * 2;     // 16 KB (experiments: widest B tile a stage holds)
constexpr int CHAIN_STAGE_BYTES = 2 * CHAIN_A_BYTES + 2 * CHAIN_B_BYTES;
constexpr int CHAIN_EPI_BYTES = CHAIN_EPI_BUFS * 2 * GEMM_BM * 64 * 2;   // hi + lo staging of 64-col chunks
constexpr int CHAIN_MAX_N = 1024;                                  // widest layer staged in smem (bias / head row)
constexpr int CHAIN_PARAM_BYTES = 2 * CHAIN_MAX_N * 4;
// ReLU mask words [buf][word][128 rows] and head partials [slice][128 rows], staged for 1-D bulk copies so
// every global write of a tile goes through the async proxy (one bulk_wait before the row-block flag)
constexpr int CHAIN_AUX_BYTES = CHAIN_EPI_BUFS * 2 * GEMM_BM * 4 + CHAIN_EPI_NQ * GEMM_BM * 4;
constexpr int CHAIN_SMEM_BYTES = 1024 + CHAIN_STAGES * CHAIN_STAGE_BYTES + CHAIN_EPI_BYTES + CHAIN_PARAM_BYTES + CHAIN_AUX_BYTES + 256;

struct ChainLayer {
  CUtensorMap a_hi, a_lo, b_hi, b_lo, c_hi, c_lo;
  // EPI_F32T: fp32 dL/dphi slabs as one 2-D map [ksplit * N rows (slab-major)][ld_f32 candidates], box
  // {128 candidates, bn features}: the tile is staged transposed in shared memory and written by one TMA
  // store (f32t_tma = 1; else per-thread stores)
  CUtensorMap c_f32;
  int f32t_tma;
  GemmArgs args;
  int epi, bn, n_tiles_n, n_tiles;     // tiles = m_tiles * n_tiles_n (n fastest)
  uint32_t idesc;
  uint32_t idesc_cat;                  // M x 2bn (FELIX_CHAIN_NCAT, CG = 1)
  // reuse: this layer's A row block is the previous layer's output and every CTA keeps its row block from
  // one layer to the next (one tile per CTA in both, same N-tile count): the CTA's own previous output
  // chunks, still in its epilogue staging buffers in the A-operand layout (128-B swizzle, K-major), serve
  // as those K blocks (no TMA load; no wait for other CTAs), issued first.
  int reuse;
  // a_exact: A is an exact 0/1 mask (fp16 hi exact, lo = 0): no A lo loads, no A lo MMA pass (the first
  // backward layer, weights prescaled by the head row); head_exact: this HEAD layer writes that mask
  int a_exact, head_exact;
  // ksplit (EPI_F32T, the last layer only): K is cut into ksplit contiguous ranges, tile = (row block, N
  // tile, part), part fastest; part p writes its partial dL/dphi to slab p of out_f32 (slab = N x ld_f32
  // floats); the reverse kernel sums the slabs in fixed order.  Spreads the largest per-CTA operand (A of
  // the K = 512 layer) over ksplit CTAs.
  int ksplit;
};

struct ChainParams {
  ChainLayer layer[CHAIN_MAX_LAYERS];
  int n_layers;
  int m_tiles;
  unsigned int* grid_bar;              // monotonic arrival counter (never reset)
  unsigned long long* trace;           // debug: [grid][layers][8] globaltimer stamps (FELIX_CHAIN_TRACE)
  // Dataflow mode (flags != nullptr): no grid barrier.  flags[(l * m_tiles + m) * 8] counts the
  // layer-l tiles of row block m whose outputs are complete (release); a layer-(l+1) tile of row block m
  // waits (acquire) until it reaches epoch * n_tiles_n(l).  Counters only grow during a search; *epoch
  // is the launch's 1-based sequence number (the forward DAG kernel's step counter, or 1 after a reset).
  unsigned int* flags;
  const int* epoch;
};

constexpr int CHAIN_FLAG_STRIDE = 8;   // one 32-B sector per counter

__device__ __forceinline__ void flag_wait(const unsigned int* f, unsigned int target) {
  unsigned int cur;
  while (true) {
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(cur) : "l"(f) : "memory");
    if (static_cast<int>(cur - target) >= 0) break;
    __nanosleep(32);
  }
}

#ifdef FELIX_CHAIN_TRACE
#define CHAIN_STAMP2(l, slot) do { unsigned long long t_; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t_)); \
    P.trace[(static_cast<size_t>(gridDim.x) * CHAIN_MAX_LAYERS + static_cast<size_t>(blockIdx.x) * CHAIN_MAX_LAYERS + (l)) * 8 + (slot)] = t_; } while (0)
#define CHAIN_STAMP(l, slot) do { unsigned long long t_; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t_)); \
    P.trace[(static_cast<size_t>(blockIdx.x) * CHAIN_MAX_LAYERS + (l)) * 8 + (slot)] = t_; } while (0)
#else
#define CHAIN_STAMP(l, slot) do {} while (0)
#define CHAIN_STAMP2(l, slot) do {} while (0)
#endif

__device__ __forceinline__ void grid_barrier(unsigned int* ctr, unsigned int nblocks) {
  // arrive (release, after this thread's async-proxy writes are complete) ...
  asm volatile("fence.proxy.async.global;" ::: "memory");
  unsigned int old;
  asm volatile("atom.add.release.gpu.u32 %0, [%1], 1;" : "=r"(old) : "l"(ctr) : "memory");
  const unsigned int target = (old / nblocks + 1) * nblocks;
  // ... and wait (acquire)
  unsigned int cur;
  do {
    asm volatile("ld.acquire.gpu.u32 %0, [%1];" : "=r"(cur) : "l"(ctr) : "memory");
  } while (static_cast<int>(cur - target) < 0);
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

// Tiles of one layer owned by this CTA (pair): tile = cluster, +#clusters, ... over all (row block
// [pair], N tile) pairs, N fastest.  CG = 1: a "pair" is one 128-row block.
template <int CG>
struct ChainTiles {
  int t0, tstep, ntn, units;
  __device__ ChainTiles(int n_tiles_n, int m_tiles, int ksplit = 1) : ntn(n_tiles_n) {
    t0 = blockIdx.x / CG;
    tstep = gridDim.x / CG;
    units = ((m_tiles + CG - 1) / CG) * ntn * ksplit;
  }
  __device__ int first() const { return t0 < units ? t0 : -1; }
  __device__ int next(int tile) const { tile += tstep; return tile < units ? tile : -1; }
};

template <int CG>
__global__ void __launch_bounds__(CHAIN_THREADS, 1) mlp_chain_kernel(const __grid_constant__ ChainParams P) {
  extern __shared__ uint8_t smem_raw[];
  // 1024-B alignment by offsetting the shared array itself (a round trip through uintptr_t would turn
  // every smem access into a generic LD/ST)
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* epi_base = smem + CHAIN_STAGES * CHAIN_STAGE_BYTES;   // [buf][hi | lo][128 x 64 fp16]
  float* s_bias = reinterpret_cast<float*>(epi_base + CHAIN_EPI_BYTES);   // [CHAIN_MAX_N] this layer's bias
  float* s_headw = s_bias + CHAIN_MAX_N;                                   // [CHAIN_MAX_N] head row (HEAD layer)
  uint32_t* s_mask = reinterpret_cast<uint32_t*>(epi_base + CHAIN_EPI_BYTES + CHAIN_PARAM_BYTES);   // [EPI_BUFS][2][128]
  float* s_cpart = reinterpret_cast<float*>(s_mask + CHAIN_EPI_BUFS * 2 * GEMM_BM);                  // [NQ][128]
  uint64_t* full_bar = reinterpret_cast<uint64_t*>(epi_base + CHAIN_EPI_BYTES + CHAIN_PARAM_BYTES + CHAIN_AUX_BYTES);
  uint64_t* empty_bar = full_bar + CHAIN_STAGES;
  uint64_t* tfull = empty_bar + CHAIN_STAGES;      // [2] accumulator ready
  uint64_t* tempty = tfull + 2;                    // [2] accumulator drained
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);
  uint32_t* gen_slot = tmem_slot + 1;              // layers completed grid-wide (producer handshake)
  uint64_t* own_bar = tempty + 4;                  // epilogue -> MMA: a tile's output chunks are staged

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const unsigned int G = gridDim.x;
  constexpr bool ncat = FELIX_CHAIN_NCAT && CG == 1;
  constexpr uint32_t ACC = ncat ? 2 * CHAIN_BN_MAX : CHAIN_BN_MAX;   // TMEM columns per accumulator buffer
  const uint32_t rank = CG == 2 ? ptx::cluster_ctarank() : 0u;

  auto a_hi = [&](int s) { return smem + s * CHAIN_STAGE_BYTES; };
  auto a_lo = [&](int s) { return smem + s * CHAIN_STAGE_BYTES + CHAIN_A_BYTES; };
  auto b_hi = [&](int s) { return smem + s * CHAIN_STAGE_BYTES + 2 * CHAIN_A_BYTES; };
  auto b_lo = [&](int s) { return smem + s * CHAIN_STAGE_BYTES + 2 * CHAIN_A_BYTES + CHAIN_B_BYTES; };

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < CHAIN_STAGES; ++s) { ptx::mbar_init(&full_bar[s], 1); ptx::mbar_init(&empty_bar[s], 1); }
    for (int a = 0; a < 2; ++a) { ptx::mbar_init(&tfull[a], 1); ptx::mbar_init(&tempty[a], CHAIN_EPI_WARPS * CG); }
    ptx::mbar_init(own_bar, CG);
    *gen_slot = 0;
    ptx::fence_barrier_init();
  }
  if (warp == 1) {
    if constexpr (CG == 2) ptx::tmem_alloc_cg2(tmem_slot, 2 * ACC);
    else ptx::tmem_alloc(tmem_slot, 2 * ACC);
  }
  ptx::tc_fence_before();
  if constexpr (CG == 2) ptx::cluster_sync();
  else __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  ptx::pdl_launch_dependents();
  ptx::pdl_wait();                                  // phi (layer-1 A operand) comes from the DAG kernel
  const bool dataflow = P.flags != nullptr;
  const unsigned int epoch = dataflow ? static_cast<unsigned int>(*reinterpret_cast<const volatile int*>(P.epoch)) : 0u;
  auto flag_of = [&](int l, int m) { return P.flags + (static_cast<size_t>(l) * P.m_tiles + m) * CHAIN_FLAG_STRIDE; };
  // leader-CTA copies of the barriers that receive arrivals from both CTAs (CG = 2)
  auto leader_addr = [&](const void* p) { return ptx::mapa_shared(ptx::smem_u32(p), 0); };
  auto arrive_leader = [&](uint64_t* bar) {
    if constexpr (CG == 2) ptx::mbar_arrive_cluster(leader_addr(bar));
    else ptx::mbar_arrive(bar);
  };
  auto wait_in = [&](uint64_t* bar, uint32_t parity) {   // barriers that receive arrivals from the peer
    if constexpr (CG == 2) ptx::mbar_wait_cluster(bar, parity);
    else ptx::mbar_wait(bar, parity);
  };
  // this CTA's 128-row block of pair tile `tile`
  auto row_block = [&](int tile, int ntn) { return (tile / ntn) * CG + static_cast<int>(rank); };

  if (warp == 0) {
    if (lane == 0) {
      // ------------------------------------------------------------ TMA producer (both CTAs)
      int it = 0;                                   // running k-block counter (ring position)
      auto load = [&](void* dst, const CUtensorMap* m, int c0, int c1, int s) {
        if constexpr (CG == 2) ptx::tma_load_2d_cg2(dst, m, c0, c1, leader_addr(&full_bar[s]));
        else ptx::tma_load_2d(dst, m, c0, c1, &full_bar[s]);
      };
      auto arm = [&](int s, uint32_t bytes_per_cta) {   // the leader expects both CTAs' bytes
        if (rank == 0) ptx::mbar_arrive_expect_tx(&full_bar[s], bytes_per_cta * CG);
      };
      for (int l = 0; l < P.n_layers; ++l) {
        const ChainLayer& L = P.layer[l];
        if (l > 0 && !dataflow) {
          // layer l reads layer l-1's outputs: wait until the epilogue warps of this CTA have
          // passed the grid barrier (they publish the layer count with st.release.cta)
          unsigned int g;
          do {
            asm volatile("ld.acquire.cta.shared::cta.u32 %0, [%1];" : "=r"(g) : "r"(ptx::smem_u32(gen_slot)) : "memory");
          } while (g < static_cast<unsigned int>(l));
          asm volatile("fence.proxy.async.global;" ::: "memory");
        }
        CHAIN_STAMP(l, 0);
        const int S = L.ksplit;
        const int nkb_all = (L.args.K + GEMM_BK - 1) / GEMM_BK;
        const int bnc = L.bn / CG;                                  // weight rows this CTA loads per tile
        // NCAT: B lo rows follow the B hi rows ([B_hi ; B_lo] is one 2bn-row operand)
        auto blo = [&](int s) { return ncat ? b_hi(s) + bnc * GEMM_BK * 2 : b_lo(s); };
        const uint32_t tx_b = 2 * (bnc * GEMM_BK * 2);
        const uint32_t tx = (L.a_exact ? 1 : 2) * CHAIN_A_BYTES + tx_b;
        ChainTiles<CG> tiles(L.n_tiles_n, P.m_tiles, S);
        for (int tile = tiles.first(); tile >= 0; tile = tiles.next(tile)) {
          const int tq = tile / S, part = tile % S;
          const int kbeg = part * nkb_all / S, nkb = (part + 1) * nkb_all / S - kbeg;
          const int mb = row_block(tq, L.n_tiles_n);
          const int m0 = mb * GEMM_BM, n0 = (tq % L.n_tiles_n) * L.bn, nb = n0 + static_cast<int>(rank) * bnc;
          int kb0 = 0;
          if (dataflow && l > 0 && L.reuse) {
            // own K blocks (B only) first, then the others (B, row-block flag once, A)
            const ChainLayer& Lp = P.layer[l - 1];
            const int own0 = (tile % Lp.n_tiles_n) * Lp.bn / GEMM_BK, nown = Lp.bn / GEMM_BK;
            bool flag_ok = false;
            for (int i = 0; i < nkb; ++i, ++it) {
              const int kb = i < nown ? own0 + i : (i - nown < own0 ? i - nown : i);
              const bool own = i < nown;
              const int s = it % CHAIN_STAGES;
              if (it >= CHAIN_STAGES) ptx::mbar_wait(&empty_bar[s], ((it / CHAIN_STAGES) - 1) & 1);
              arm(s, own ? tx_b : tx);
              load(b_hi(s), &L.b_hi, kb * GEMM_BK, nb, s);
              load(blo(s), &L.b_lo, kb * GEMM_BK, nb, s);
              if (!own) {
                if (!flag_ok) {
                  flag_wait(flag_of(l - 1, mb), epoch * static_cast<unsigned int>(Lp.n_tiles_n));
                  asm volatile("fence.proxy.async.global;" ::: "memory");
                  flag_ok = true;
                  if (tile == tiles.first()) CHAIN_STAMP(l, 5);
                }
                load(a_hi(s), &L.a_hi, kb * GEMM_BK, m0, s);
                if (!L.a_exact) load(a_lo(s), &L.a_lo, kb * GEMM_BK, m0, s);
              }
            }
            continue;
          }
          if (dataflow && l > 0) {
            // weights do not depend on the previous layer: put the first ring stages' B loads in flight,
            // then wait for this row block of layer l-1 and add the A loads
            const int pre = nkb < CHAIN_STAGES ? nkb : CHAIN_STAGES;
            for (int kb = 0; kb < pre; ++kb) {
              const int s = (it + kb) % CHAIN_STAGES;
              if (it + kb >= CHAIN_STAGES) ptx::mbar_wait(&empty_bar[s], (((it + kb) / CHAIN_STAGES) - 1) & 1);
              arm(s, tx);
              load(b_hi(s), &L.b_hi, (kbeg + kb) * GEMM_BK, nb, s);
              load(blo(s), &L.b_lo, (kbeg + kb) * GEMM_BK, nb, s);
            }
            flag_wait(flag_of(l - 1, mb), epoch * static_cast<unsigned int>(P.layer[l - 1].n_tiles_n));
            asm volatile("fence.proxy.async.global;" ::: "memory");
            if (tile == tiles.first()) CHAIN_STAMP(l, 5);
            for (int kb = 0; kb < pre; ++kb) {
              const int s = (it + kb) % CHAIN_STAGES;
              load(a_hi(s), &L.a_hi, (kbeg + kb) * GEMM_BK, m0, s);
              if (!L.a_exact) load(a_lo(s), &L.a_lo, (kbeg + kb) * GEMM_BK, m0, s);
            }
            kb0 = pre;
            it += pre;
          }
          for (int kb = kb0; kb < nkb; ++kb, ++it) {
            const int s = it % CHAIN_STAGES;
            if (it >= CHAIN_STAGES) ptx::mbar_wait(&empty_bar[s], ((it / CHAIN_STAGES) - 1) & 1);
            arm(s, tx);
            const int k0 = (kbeg + kb) * GEMM_BK;
            load(a_hi(s), &L.a_hi, k0, m0, s);
            if (!L.a_exact) load(a_lo(s), &L.a_lo, k0, m0, s);
            load(b_hi(s), &L.b_hi, k0, nb, s);
            load(blo(s), &L.b_lo, k0, nb, s);
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && rank == 0) {
      // ------------------------------------------------------------ MMA issuer (leader CTA)
      int it = 0, tcount = 0;
      int staged_tiles = 0, chunk_count = 0, prev_chunk_base = 0;   // mirror of the epilogue's staging sequence
      for (int l = 0; l < P.n_layers; ++l) {
        const ChainLayer& L = P.layer[l];
        const int S = L.ksplit;
        const int nkb_all = (L.args.K + GEMM_BK - 1) / GEMM_BK;
        ChainTiles<CG> tiles(L.n_tiles_n, P.m_tiles, S);
        for (int tile = tiles.first(); tile >= 0; tile = tiles.next(tile), ++tcount) {
          const int part = tile % S;
          const int nkb = (part + 1) * nkb_all / S - part * nkb_all / S;
          const int acc = tcount & 1;
          if (tcount >= 2) wait_in(&tempty[acc], ((tcount >> 1) - 1) & 1);
          ptx::tc_fence_after();
          const uint32_t d = tmem_base + acc * ACC;
          const bool reuse = dataflow && l > 0 && L.reuse;
          const bool a_exact = L.a_exact != 0;
          int own0 = 0, nown = 0;
          if (reuse) {
            const ChainLayer& Lp = P.layer[l - 1];
            own0 = (tile % Lp.n_tiles_n) * Lp.bn / GEMM_BK;
            nown = Lp.bn / GEMM_BK;
            // the previous tile's chunks are staged (in both CTAs) and fenced for the async proxy
            wait_in(own_bar, (staged_tiles - 1) & 1);
          }
          for (int i = 0; i < nkb; ++i, ++it) {
            const int kb = !reuse ? i : (i < nown ? own0 + i : (i - nown < own0 ? i - nown : i));
            (void)kb;
            const int s = it % CHAIN_STAGES;
            wait_in(&full_bar[s], (it / CHAIN_STAGES) & 1);
            if (i == 0 && tcount == 0) CHAIN_STAMP(l, 1);
            ptx::tc_fence_after();
            uint32_t ah = ptx::smem_u32(a_hi(s)), al = ptx::smem_u32(a_lo(s));
            if (reuse && i < nown) {
              const uint8_t* eh = epi_base + ((prev_chunk_base + i) % CHAIN_EPI_BUFS) * (2 * GEMM_BM * 64 * 2);
              ah = ptx::smem_u32(eh);
              al = ptx::smem_u32(eh + GEMM_BM * 64 * 2);
            }
            const uint32_t bh = ptx::smem_u32(b_hi(s)), bl = ptx::smem_u32(b_lo(s));
#pragma unroll
            for (int kk = 0; kk < GEMM_BK / GEMM_UMMA_K; ++kk) {
              const uint32_t off = kk * GEMM_UMMA_K * 2;
              const uint32_t acc0 = (i | kk) != 0;
              if constexpr (ncat) {
                // [A_hi x B_hi | A_hi x B_lo] in columns [0, 2bn), then A_lo x B_hi into [0, bn)
                ptx::mma_f16_ss(d, ptx::sdesc_k_sw128(ah + off), ptx::sdesc_k_sw128(bh + off), L.idesc_cat, acc0);
                if (!a_exact) ptx::mma_f16_ss(d, ptx::sdesc_k_sw128(al + off), ptx::sdesc_k_sw128(bh + off), L.idesc, 1u);
              } else if constexpr (CG == 2) {
                if (!a_exact) ptx::mma_f16_ss_cg2(d, ptx::sdesc_k_sw128(al + off), ptx::sdesc_k_sw128(bh + off), L.idesc, acc0);
                ptx::mma_f16_ss_cg2(d, ptx::sdesc_k_sw128(ah + off), ptx::sdesc_k_sw128(bl + off), L.idesc, a_exact ? acc0 : 1u);
                ptx::mma_f16_ss_cg2(d, ptx::sdesc_k_sw128(ah + off), ptx::sdesc_k_sw128(bh + off), L.idesc, 1u);
              } else {
                if (!a_exact) ptx::mma_f16_ss(d, ptx::sdesc_k_sw128(al + off), ptx::sdesc_k_sw128(bh + off), L.idesc, acc0);
                ptx::mma_f16_ss(d, ptx::sdesc_k_sw128(ah + off), ptx::sdesc_k_sw128(bl + off), L.idesc, a_exact ? acc0 : 1u);
                ptx::mma_f16_ss(d, ptx::sdesc_k_sw128(ah + off), ptx::sdesc_k_sw128(bh + off), L.idesc, 1u);
              }
            }
            if constexpr (CG == 2) ptx::mma_commit_mc(&empty_bar[s], 0x3);
            else ptx::mma_commit(&empty_bar[s]);
          }
          if constexpr (CG == 2) ptx::mma_commit_mc(&tfull[acc], 0x3);
          else ptx::mma_commit(&tfull[acc]);
          CHAIN_STAMP(l, 2);
          if (L.epi != EPI_F32T) {          // the epilogue will stage this tile's bn / 64 chunks
            prev_chunk_base = chunk_count;
            chunk_count += L.bn / 64;
            // own_bar completes one phase per tile whose chunks the NEXT layer reuses (every arrive is waited on)
            if (dataflow && l + 1 < P.n_layers && P.layer[l + 1].reuse) ++staged_tiles;
          }
        }
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue warps 2.. (both CTAs)
    constexpr int CPW = CHAIN_EPI_CPW, NQ = CHAIN_EPI_NQ;
    const int q = warp & 3;                          // TMEM lane quadrant this warp may access
    const int sub = (warp - 2) >> 2;                 // which CPW-column slice of each 64-column chunk
    const int cs = sub * CPW;
    const int r_tile = q * 32 + lane;
    const int etid = threadIdx.x - 64;
    int epi_count = 0;                               // 64-column chunks staged so far (buffer parity)
    constexpr int NEPI = CHAIN_EPI_WARPS * 32;
    int tcount = 0;
    // CPW accumulator columns c .. c+CPW-1 of this thread's row (NCAT: the two halves summed)
    auto acc_cols = [&](uint32_t t_row, int c, int bn, float (&v)[CPW]) {
      if constexpr (ncat) {
#pragma unroll
        for (int h = 0; h < CPW; h += 16) {
          float t[32];
          ptx::tmem_ld2x16(t_row + c + h, t_row + bn + c + h, t);
#pragma unroll
          for (int i = 0; i < 16; ++i) v[h + i] = t[i] + t[16 + i];
        }
      } else if constexpr (CPW == 32) {
        float t[32];
        ptx::tmem_ld2x16(t_row + c, t_row + c + 16, t);
#pragma unroll
        for (int i = 0; i < 32; ++i) v[i] = t[i];
      } else {
        float t[16];
        ptx::tmem_ld16(t_row + c, t);
#pragma unroll
        for (int i = 0; i < 16; ++i) v[i] = t[i];
      }
    };
    for (int l = 0; l < P.n_layers; ++l) {
      const ChainLayer& L = P.layer[l];
      // per-layer fields in registers once: read through the dynamically indexed param block, the
      // compiler otherwise re-fetches each pointer (LDC) before every element access
      const int epi = L.epi, bn = L.bn, ntn = L.n_tiles_n;
      const bool hexact = L.head_exact != 0;   // HEAD: write the 0/1 mask (the next layer's weights carry -w)
      const int aM = L.args.M, n_valid = L.args.n_valid, ld_f32 = L.args.ld_f32, ld_c = L.args.ld_c;
      const int aN = L.args.N;
      const int ld_mask = L.args.ld_mask;
      const float* __restrict__ bias = L.args.bias;
      const float* __restrict__ head_w = L.args.head_w;
      uint32_t* __restrict__ mask_out = L.args.mask_out;
      const uint32_t* mask_in = L.args.mask_in;
      float* __restrict__ c_part = L.args.c_part;
      float* __restrict__ out_f32 = L.args.out_f32;
      const CUtensorMap* tm_c_hi = &L.c_hi;
      const CUtensorMap* tm_c_lo = &L.c_lo;
      const bool next_reuse = dataflow && l + 1 < P.n_layers && P.layer[l + 1].reuse;
      const int S = L.ksplit;
      // stage this layer's bias / head row in smem while the MMA warp works (previous layer's
      // readers are past the layer-end barrier, so the buffer is free)
      if (epi == EPI_RELU || epi == EPI_HEAD) {
        for (int i = etid; i < aN; i += NEPI) {
          s_bias[i] = __ldg(&bias[i]);
          if (epi == EPI_HEAD) s_headw[i] = __ldg(&head_w[i]);
        }
      }
      ptx::named_bar_sync(1, NEPI);
      ChainTiles<CG> tiles(ntn, P.m_tiles, S);
      const int first_tile = tiles.first();
      for (int tile = first_tile; tile >= 0; tile = tiles.next(tile), ++tcount) {
        const int acc = tcount & 1;
        const int tq = tile / S, part = tile % S;
        const int mb = row_block(tq, ntn);
        const int m0 = mb * GEMM_BM, n0 = (tq % ntn) * bn;
        const int row = m0 + r_tile;
        const bool row_ok = row < aM;
        // this thread's mask bits for the tile (<= 2 chunks of 64 columns), requested before the wait
        uint32_t mwords[CHAIN_BN_MAX / 64] = {0u};
        if (dataflow && epi == EPI_MASK) {
          // the mask words come from an earlier layer of this row block (other CTAs): acquire the
          // row block's flag of the previous layer first (the epilogue warps are idle in the mainloop)
          if (etid == 0) flag_wait(flag_of(l - 1, mb), epoch * static_cast<unsigned int>(P.layer[l - 1].n_tiles_n));
          ptx::named_bar_sync(1, NEPI);
        }
        if (epi == EPI_MASK && row_ok) {
          // written earlier in this launch by other CTAs: coherent L2 load, not the .nc path
#pragma unroll
          for (int q64 = 0; q64 < CHAIN_BN_MAX / 64; ++q64)
            if (q64 * 64 < bn) mwords[q64] = __ldcg(&mask_in[static_cast<size_t>((n0 + q64 * 64 + cs) / 32) * ld_mask + row]) >> (cs & 31);
        }
        ptx::mbar_wait(&tfull[acc], (tcount >> 1) & 1);
        if (etid == 0 && tile == first_tile) CHAIN_STAMP(l, 3);
        ptx::tc_fence_after();
        const uint32_t t_row = tmem_base + acc * ACC + (static_cast<uint32_t>(q * 32) << 16);
        float head_acc = 0.f;
        if (epi == EPI_F32T && L.f32t_tma) {
          // stage [bn features][128 rows] fp32 (48 KB at bn = 96, in the epilogue staging buffers: the last
          // layer, nothing reuses them), then one TMA store of the tile into slab `part`
          float* stg = reinterpret_cast<float*>(epi_base);
          if (etid == 0) ptx::bulk_wait_read<0>();          // a previous tile's store has read the staging
          ptx::named_bar_sync(1, NEPI);
          for (int c = cs; c < bn; c += 64) {
            float v[CPW];
            acc_cols(t_row, c, bn, v);
#pragma unroll
            for (int i = 0; i < CPW; ++i)
              if (c + i < bn) stg[(c + i) * GEMM_BM + r_tile] = v[i];
          }
          ptx::fence_proxy_async_smem();
          ptx::named_bar_sync(1, NEPI);
          if (etid == 0) {
            asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
                         :: "l"(reinterpret_cast<uint64_t>(&L.c_f32)), "r"(m0), "r"(part * aN + n0), "r"(ptx::smem_u32(stg)) : "memory");
            ptx::bulk_commit();
          }
        } else if (epi == EPI_F32T) {
          for (int c = cs; c < bn; c += 64) {
            float v[CPW];
            acc_cols(t_row, c, bn, v);
            const int n = n0 + c;
            float* __restrict__ slab = out_f32 + static_cast<size_t>(part) * aN * ld_f32;
            if (row_ok) {
#pragma unroll
              for (int i = 0; i < CPW; ++i)
                if (n + i < n_valid) slab[static_cast<size_t>(n + i) * ld_f32 + row] = v[i];
            }
          }
        } else {
          for (int c64 = 0; c64 < bn; c64 += 64) {
            // the staging buffer must be free: the TMA store that last used it finished reading
            const int ebuf = epi_count % CHAIN_EPI_BUFS;
            uint8_t* epi_hi = epi_base + ebuf * (2 * GEMM_BM * 64 * 2);
            uint8_t* epi_lo = epi_hi + GEMM_BM * 64 * 2;
            ++epi_count;
            if (etid == 0) {
              if (CHAIN_EPI_BUFS == 2) ptx::bulk_wait_read<1>(); else ptx::bulk_wait_read<0>();
            }
            ptx::named_bar_sync(1, NEPI);
            const bool st0 = etid == 0 && c64 == 0 && tile == first_tile;
            if (st0) CHAIN_STAMP2(l, 0);
            {
              const int c = c64 + cs;
              float v[CPW];
              acc_cols(t_row, c, bn, v);
              if (st0) CHAIN_STAMP2(l, 1);
              const int n = n0 + c;
              if (epi == EPI_MASK) {
                const uint32_t bits = c64 == 0 ? mwords[0] : mwords[CHAIN_BN_MAX / 64 - 1];
#pragma unroll
                for (int i = 0; i < CPW; ++i) v[i] = ((bits >> i) & 1u) ? v[i] : 0.f;
              } else {
                uint32_t bits = 0;
                const bool head = epi == EPI_HEAD;
                // two separate loops: a runtime `head` inside one loop is if-converted, so ReLU layers would
                // execute the head arithmetic too (~16 instead of ~8 instructions per element)
                if (!head) {
#pragma unroll
                  for (int i4 = 0; i4 < CPW; i4 += 4) {
                    const float4 b4 = *reinterpret_cast<const float4*>(s_bias + n + i4);
                    const float bb[4] = {b4.x, b4.y, b4.z, b4.w};
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                      const int i = i4 + u;
                      const float z = v[i] + bb[u];
                      const bool on = z > 0.f;
                      bits |= (on ? 1u : 0u) << i;
                      v[i] = on ? z : 0.f;
                    }
                  }
                } else {
#pragma unroll
                  for (int i4 = 0; i4 < CPW; i4 += 4) {
                    const float4 b4 = *reinterpret_cast<const float4*>(s_bias + n + i4);
                    const float4 w4 = *reinterpret_cast<const float4*>(s_headw + n + i4);
                    const float bb[4] = {b4.x, b4.y, b4.z, b4.w}, ww[4] = {w4.x, w4.y, w4.z, w4.w};
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                      const int i = i4 + u;
                      const float z = v[i] + bb[u];
                      const bool on = z > 0.f;
                      head_acc += (on ? z : 0.f) * ww[u];
                      v[i] = on ? (hexact ? 1.f : -ww[u]) : 0.f;   // delta_{L-1} = W_L^T (dL/dc = -1) (.) [Z > 0]
                    }
                  }
                }
                if (!head) {
                  uint32_t* mw = s_mask + (ebuf * 2 + cs / 32) * GEMM_BM + r_tile;   // word (n0 + c64 + cs) / 32 of the row
                  if constexpr (CPW == 32) *mw = bits;
                  else reinterpret_cast<uint16_t*>(mw)[(cs >> 4) & 1] = static_cast<uint16_t>(bits);
                }
              }
#pragma unroll
              for (int qq = 0; qq < CPW / 8; ++qq) {
                // split 8 values into fp16 hi / lo with packed f16x2 converts
                uint32_t h[4], lo[4];
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                  const float2 f = make_float2(v[qq * 8 + 2 * u], v[qq * 8 + 2 * u + 1]);
                  const __half2 hh = __float22half2_rn(f);
                  const float2 back = __half22float2(hh);
                  const __half2 ll = __float22half2_rn(make_float2(f.x - back.x, f.y - back.y));
                  h[u] = *reinterpret_cast<const uint32_t*>(&hh);
                  lo[u] = *reinterpret_cast<const uint32_t*>(&ll);
                }
                const int q16 = cs / 8 + qq;
                const uint32_t off = r_tile * 128 + ((q16 ^ (r_tile & 7)) << 4);
                *reinterpret_cast<uint4*>(epi_hi + off) = make_uint4(h[0], h[1], h[2], h[3]);
                if (!hexact) *reinterpret_cast<uint4*>(epi_lo + off) = make_uint4(lo[0], lo[1], lo[2], lo[3]);
              }
            }
            if (st0) CHAIN_STAMP2(l, 2);
            ptx::fence_proxy_async_smem();
            ptx::named_bar_sync(1, NEPI);
            if (st0) CHAIN_STAMP2(l, 3);
            if (etid == 0) {
              ptx::tma_store_2d(tm_c_hi, n0 + c64, m0, epi_hi);
              if (!hexact) ptx::tma_store_2d(tm_c_lo, n0 + c64, m0, epi_lo);   // exact mask: lo = 0, never read
              if (epi == EPI_RELU) {   // the chunk's two mask-word columns (rows m0 .. m0+127; ld_mask >= padded rows)
                ptx::bulk_s2g(mask_out + static_cast<size_t>((n0 + c64) / 32) * ld_mask + m0, s_mask + (ebuf * 2) * GEMM_BM, GEMM_BM * 4);
                ptx::bulk_s2g(mask_out + static_cast<size_t>((n0 + c64) / 32 + 1) * ld_mask + m0, s_mask + (ebuf * 2 + 1) * GEMM_BM, GEMM_BM * 4);
              }
              ptx::bulk_commit();
              if (c64 + 64 >= bn && next_reuse) arrive_leader(own_bar);   // all chunks staged, the next layer reuses them
            }
          }
        }
        // head partial per (N tile, column slice); the reverse kernel sums all NQ * N / bn partials.  Staged in
        // shared memory and bulk-copied (rows m0 .. m0+127; c_part has padded rows)
        if (epi == EPI_HEAD) {
          if (etid == 0) ptx::bulk_wait_read<0>();          // the previous tile's copy has read s_cpart
          ptx::named_bar_sync(1, NEPI);
          s_cpart[sub * GEMM_BM + r_tile] = head_acc;
          ptx::fence_proxy_async_smem();
          ptx::named_bar_sync(1, NEPI);
          if (etid == 0) {
#pragma unroll
            for (int j = 0; j < NQ; ++j)
              ptx::bulk_s2g(c_part + static_cast<size_t>(NQ * (n0 / bn) + j) * ld_c + m0, s_cpart + j * GEMM_BM, GEMM_BM * 4);
            ptx::bulk_commit();
          }
        }
        // accumulator drained: let the (leader's) MMA warp reuse it
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) arrive_leader(&tempty[acc]);
        if (dataflow && l + 1 < P.n_layers && etid == 0) {
          // every global write of this tile (activations, mask words, head partials) was a bulk copy issued
          // by this thread: complete them, then count the tile (release)
          ptx::bulk_wait<0>();
          asm volatile("fence.proxy.async.global;" ::: "memory");
          asm volatile("red.release.gpu.global.add.u32 [%0], 1;" :: "l"(flag_of(l, mb)) : "memory");
          if (tile == first_tile) CHAIN_STAMP(l, 6);
        }
      }
      // ---- layer end: all of this CTA's outputs complete + visible, then the grid barrier
      if (etid == 0) CHAIN_STAMP(l, 4);
      if (l + 1 < P.n_layers && !dataflow) {
        if (etid == 0) ptx::bulk_wait<0>();
        __threadfence();
        ptx::named_bar_sync(1, NEPI);
        if (etid == 0) {
          CHAIN_STAMP(l, 5);
          grid_barrier(P.grid_bar, G);
          CHAIN_STAMP(l, 6);
          // publish "layer l done everywhere" to the producer warp of this CTA
          asm volatile("st.release.cta.shared::cta.u32 [%0], %1;" :: "r"(ptx::smem_u32(gen_slot)), "r"(static_cast<unsigned int>(l + 1)) : "memory");
        }
      }
    }
    if (etid == 0) ptx::bulk_wait<0>();
  }
  ptx::tc_fence_before();
  if constexpr (CG == 2) ptx::cluster_sync();
  else __syncthreads();
  if (warp == 1) {
    if constexpr (CG == 2) ptx::tmem_dealloc_cg2(tmem_base, 2 * ACC);
    else ptx::tmem_dealloc(tmem_base, 2 * ACC);
  }
}

}  // namespace felix
