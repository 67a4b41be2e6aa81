// felix_api.cu — libfelix: the C ABI of include/felix.h on B200 (sm_100a).
//
// Per search step (Algorithm 1 lines 16-19) the device runs, with no host round trip:
//   felix_fwd (NVRTC, per space)  ->  L-1 forward tcgen05 GEMMs  ->  L-1 backward tcgen05 GEMMs
//   ->  felix_rev_adam (NVRTC, per space)
// and after the search (lines 20-21): rounding (K5), hard features + validity (NVRTC), FP64 MLP
// scoring (K6), dedup + top-k (K7).
#include <algorithm>
#include <atomic>
#include <set>
#include <chrono>
#include <cmath>
#include <cstring>
#include <cstdlib>
#include <functional>
#include <map>
#include <mutex>
#include <numeric>
#include <string>
#include <thread>
#include <memory>
#include <vector>
#include <nvrtc.h>
#include <cudaTypedefs.h>
#include "felix_internal.h"
#include "mlp_gemm.cuh"
#include "mlp_chain.cuh"
#include "mlp_tile.cuh"
#include "aux_kernels.cuh"

namespace felix {

static thread_local std::string g_last_error;
void set_error(const std::string& m) { g_last_error = m; }

uint64_t next_uid() {
  static std::atomic<uint64_t> ctr{1};
  return ctr.fetch_add(1);
}

// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) is per device context: remember (kernel, device)
// pairs already configured, under a mutex (concurrent callers, several GPUs in one process).
static void set_smem_attr(const void* fn, int bytes, bool nonportable_cluster = false) {
  static std::mutex mu;
  static std::set<std::pair<const void*, int>> done;
  int dev = 0;
  CUDA_OK(cudaGetDevice(&dev));
  std::lock_guard<std::mutex> lk(mu);
  if (done.count({fn, dev})) return;
  CUDA_OK(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes));
  if (nonportable_cluster) CUDA_OK(cudaFuncSetAttribute(fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 0));
  done.insert({fn, dev});
}

// ============================================================================ GEMM dispatch
struct GemmLaunch {
  int epi = 0, bn = 0, stages = 2;
  CUtensorMap a_hi, a_lo, b_hi, b_lo, c_hi, c_lo;   // c: output tiles (TMA store), = next GEMM's A maps
  const void* w_hi = nullptr;                         // B operand (weights) base pointers
  const void* w_lo = nullptr;
  GemmArgs args{};
  dim3 grid;
};

// Programmatic dependent launch: the kernel's prologue (barrier init, TMEM alloc, descriptor
// prefetch) overlaps the previous kernel's tail; griddepcontrol.wait orders the data accesses.
static cudaLaunchAttribute g_pdl_attr = [] {
  cudaLaunchAttribute a{};
  a.id = cudaLaunchAttributeProgrammaticStreamSerialization;
  a.val.programmaticStreamSerializationAllowed = 1;
  return a;
}();

static int pdl_mask();   // felix_tune("pdl") below

template <int BN, int EPI>
static void launch_gemm_t(const GemmLaunch& g, cudaStream_t st) {
  auto kern = mlp_gemm_kernel<BN, EPI>;
  set_smem_attr(reinterpret_cast<const void*>(kern), GemmCfg<BN>::smem_bytes(GemmCfg<BN>::MAX_STAGES));
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = g.grid;
  cfg.blockDim = dim3(128);
  cfg.dynamicSmemBytes = GemmCfg<BN>::smem_bytes(g.stages);
  cfg.stream = st;
  cfg.attrs = &g_pdl_attr;
  cfg.numAttrs = (pdl_mask() & 2) ? 1 : 0;
  CUDA_OK(cudaLaunchKernelEx(&cfg, kern, g.a_hi, g.a_lo, g.b_hi, g.b_lo, g.c_hi, g.c_lo, g.args, g.stages));
}

static int gemm_max_stages(int bn) {
  switch (bn) {
    case 64: return GemmCfg<64>::MAX_STAGES;
    case 96: return GemmCfg<96>::MAX_STAGES;
    case 128: return GemmCfg<128>::MAX_STAGES;
    default: return GemmCfg<256>::MAX_STAGES;
  }
}

static void launch_gemm(const GemmLaunch& g, cudaStream_t st) {
#define FELIX_G(BN_, EPI_) if (g.bn == BN_ && g.epi == EPI_) return launch_gemm_t<BN_, EPI_>(g, st)
  FELIX_G(64, EPI_RELU); FELIX_G(128, EPI_RELU); FELIX_G(256, EPI_RELU);
  FELIX_G(64, EPI_HEAD); FELIX_G(128, EPI_HEAD); FELIX_G(256, EPI_HEAD);
  FELIX_G(64, EPI_MASK); FELIX_G(128, EPI_MASK); FELIX_G(256, EPI_MASK);
  FELIX_G(64, EPI_F32T); FELIX_G(96, EPI_F32T); FELIX_G(128, EPI_F32T); FELIX_G(256, EPI_F32T);
#undef FELIX_G
  FELIX_THROW(FELIX_E_UNSUPPORTED, "no GEMM instantiation for BN=" + std::to_string(g.bn));
}

// cuTensorMapEncodeTiled through the runtime's driver entry point: libfelix does not link libcuda,
// so it loads (and its symbols can be inspected) on a machine without a GPU driver.
static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    CUDA_OK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q));
    if (q != cudaDriverEntryPointSuccess || !p) FELIX_THROW(FELIX_E_CUDA, "cuTensorMapEncodeTiled unavailable");
    fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  }
  return fn;
}

static CUtensorMap make_tmap(const void* base, int64_t rows, int64_t cols, int box_rows) {
  CUtensorMap m;
  cuuint64_t dims[2] = {static_cast<cuuint64_t>(cols), static_cast<cuuint64_t>(rows)};
  cuuint64_t strides[1] = {static_cast<cuuint64_t>(cols) * 2};
  cuuint32_t box[2] = {static_cast<cuuint32_t>(GEMM_BK), static_cast<cuuint32_t>(box_rows)};
  cuuint32_t es[2] = {1, 1};
  CU_OK(encode_fn()(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void*>(base), dims, strides, box, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                               CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE));
  return m;
}

// fp32 [rows][cols] row-major (cols contiguous), no swizzle, box {box_cols (inner), box_rows}
static CUtensorMap make_tmap_f32(const void* base, int64_t rows, int64_t cols, int box_cols, int box_rows) {
  CUtensorMap m;
  cuuint64_t dims[2] = {static_cast<cuuint64_t>(cols), static_cast<cuuint64_t>(rows)};
  cuuint64_t strides[1] = {static_cast<cuuint64_t>(cols) * 4};
  cuuint32_t box[2] = {static_cast<cuuint32_t>(box_cols), static_cast<cuuint32_t>(box_rows)};
  cuuint32_t es[2] = {1, 1};
  CU_OK(encode_fn()(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<void*>(base), dims, strides, box, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                               CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE));
  return m;
}

// ============================================================================ execution knobs
// Process-wide knobs set through felix_tune (experiments and tests only; the library never reads the
// environment).  -1 = the measured default.
struct Tuning {
  std::atomic<int> mlp{-1};          // 0 tile kernel, 1 persistent chain, 2 per-layer GEMMs
  std::atomic<int> P{-1};            // cone-partition width of the DAG kernels
  std::atomic<int> R{-1};            // replicas of the cone groups per block
  std::atomic<int> scw{-1};          // warps per split-cone reverse CTA
  std::atomic<int> chunks{-1};       // concurrent population chunks
  std::atomic<int> sc{-1};           // split-cone reverse kernel (1) or cone-group kernel (0)
  std::atomic<int> tile_cg{-1};      // tile kernel: 1-SM tiles (1) or 2-SM cta_group::2 pairs (2)
  std::atomic<int> chain_cg{-1};     // layer chain: 1-SM tiles (1) or 2-SM cta_group::2 pairs (2)
  std::atomic<int> dphi_ksplit{-1};  // layer chain: split-K parts of the dL/dphi layer (1, 2, 4)
  std::atomic<int> codegen_P{-1}, codegen_R{-1};   // felix_codegen's variant
  std::atomic<int> trace{0};         // per-block %globaltimer stamps in kernels generated afterwards
  std::atomic<int> round_bnb{0};
  std::atomic<int> graph_steps{-1};  // Adam steps per search graph (-1: kGraphSteps)
  std::atomic<int> score_dmma{-1};  // FP64 scoring layers on the FP64 tensor cores (0: CUDA-core kernel; -1 = 1)
  std::atomic<int> dphi_tma{-1};     // chain dL/dphi epilogue: one TMA store per tile (1, default) or per-thread stores (0)
  std::atomic<int> pdl{-1};          // PDL edges: bit 0 forward, 1 MLP kernels, 2 reverse / other (-1: none)     // 1: every split component rounds by branch and bound (test hook)
};
static Tuning g_tune;

// ============================================================================ per-(space, model, n) plan
struct Plan {
  const CostModel* cm = nullptr;
  int64_t n = -1, n_pad = 0;
  DevBuf phi_hi, phi_lo;                                   // [n][K0p]
  std::vector<std::unique_ptr<DevBuf>> act_hi, act_lo, mask;  // per hidden layer l = 1..L-1
  DevBuf c_part, dphi, m, v, step_ctr;
  int dphi_parts = 1;                      // split-K slabs of dL/dphi the reverse kernel sums (chain only)
  DevBuf sc_part, sc_pen;                                // split-cone reverse: partial adjoints, penalties
  int n_head_tiles = 0;
  std::vector<GemmLaunch> gemms;           // per-layer kernels (FELIX_MLP=layers)
  ChainParams chain{};                     // persistent all-layer kernel
  int chain_grid = 0;
  int chain_cg = 1;                        // 2: 2-SM cta_group::2 pairs (256-row tiles, weights split along N)
  DevBuf grid_bar;
  DevBuf chain_flags;                      // dataflow chain: per (layer, row block) completion counters
  bool tile_ok = false;                    // model has the shape mlp_tile_kernel is specialised for
  TileParams tile{};                       // tile-local fused MLP (default when tile_ok)
  int tile_grid = 0;
  int tile_cg = 1;                         // 1 = one SM per 128-row tile; 2 = 2-SM cta_group::2 pairs (felix_tune)
  bool tile_full_wave = false;             // >= one 128-row tile per SM
  int mode = 0;                            // MlpMode, fixed when the plan is built
};

// MLP execution mode: "tile" (tile-local fused kernel), "chain" (persistent layer-by-layer kernel),
// "layers" (one kernel per GEMM).  felix_tune("mlp") overrides.  Default (measured on B200, DESIGN.md
// "MLP modes"): a tile's serial on-chip pipeline takes ~55 us whatever the population, so the tile
// kernel wins once there is at least one full wave of 128-row tiles (C5 shard: 364 vs 518 us per
// Adam step) and the chain, which spreads every layer over all SMs, wins below that (C2: 48 vs 56 us).
enum MlpMode { MLP_TILE, MLP_CHAIN, MLP_LAYERS };
static MlpMode mlp_mode(const Plan& p) {
  const int t = g_tune.mlp.load();
  if (t == 2) return MLP_LAYERS;
  if (t == 1) return MLP_CHAIN;
  if (t == 0 && p.tile_ok) return MLP_TILE;
  return (p.tile_ok && p.tile_full_wave) ? MLP_TILE : MLP_CHAIN;
}
static bool use_chain() { return g_tune.mlp.load() != 2; }
// Programmatic dependent launch edges (felix_tune "pdl", bit mask: 1 forward DAG kernel, 2 MLP kernels,
// 4 reverse / other kernels).  Default none: measured at C2 (profiles/r02/bench_pdl.log), every edge costs
// more than the prologue overlap it buys -- the early-resident dependent CTAs slow the running kernel
// (no PDL 8.75e7 cand-steps/s; chain + reverse edges 8.22e7; all edges 7.74e7).
static int pdl_mask() { const int m = g_tune.pdl.load(); return m >= 0 ? m : 0; }

static void launch_tile(const Plan& p, cudaStream_t st) {
  const void* fn = p.tile_cg == 2 ? reinterpret_cast<const void*>(mlp_tile_kernel<2>)
                                  : reinterpret_cast<const void*>(mlp_tile_kernel<1>);
  set_smem_attr(fn, tile::SMEM_BYTES, p.tile_cg == 2);
  cudaLaunchAttribute attrs[2];
  attrs[0] = g_pdl_attr;
  if (!(pdl_mask() & 2)) attrs[0].val.programmaticStreamSerializationAllowed = 0;
  attrs[1].id = cudaLaunchAttributeClusterDimension;
  attrs[1].val.clusterDim.x = static_cast<unsigned>(p.tile_cg);
  attrs[1].val.clusterDim.y = 1;
  attrs[1].val.clusterDim.z = 1;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(static_cast<unsigned>(p.tile_grid));
  cfg.blockDim = dim3(tile::THREADS);
  cfg.dynamicSmemBytes = tile::SMEM_BYTES;
  cfg.stream = st;
  cfg.attrs = attrs;
  cfg.numAttrs = p.tile_cg == 2 ? 2 : 1;
  if (p.tile_cg == 2) CUDA_OK(cudaLaunchKernelEx(&cfg, mlp_tile_kernel<2>, p.tile));
  else CUDA_OK(cudaLaunchKernelEx(&cfg, mlp_tile_kernel<1>, p.tile));
}

static void launch_chain(const Plan& p, cudaStream_t st) {
  const bool cg2 = p.chain_cg == 2;
  set_smem_attr(cg2 ? reinterpret_cast<const void*>(mlp_chain_kernel<2>) : reinterpret_cast<const void*>(mlp_chain_kernel<1>),
                CHAIN_SMEM_BYTES);
  cudaLaunchAttribute attrs[3];
  attrs[0] = g_pdl_attr;
  if (!(pdl_mask() & 2)) attrs[0].val.programmaticStreamSerializationAllowed = 0;
  attrs[1].id = cudaLaunchAttributeCooperative;   // the dataflow flags need every CTA resident
  attrs[1].val.cooperative = 1;
  attrs[2].id = cudaLaunchAttributeClusterDimension;
  attrs[2].val.clusterDim.x = 2;
  attrs[2].val.clusterDim.y = 1;
  attrs[2].val.clusterDim.z = 1;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(static_cast<unsigned>(p.chain_grid));
  cfg.blockDim = dim3(CHAIN_THREADS);
  cfg.dynamicSmemBytes = CHAIN_SMEM_BYTES;
  cfg.stream = st;
  cfg.attrs = attrs;
  cfg.numAttrs = cg2 ? 3 : 2;
  if (cg2) CUDA_OK(cudaLaunchKernelEx(&cfg, mlp_chain_kernel<2>, p.chain));
  else CUDA_OK(cudaLaunchKernelEx(&cfg, mlp_chain_kernel<1>, p.chain));
}

// The population split into K independent chunks, each with its own workspace (Plan).  One Adam
// step of all chunks is captured as ONE CUDA graph with K parallel branches (fork/join), so one
// chunk's tensor-core GEMMs overlap another chunk's latency-bound expression kernels.
constexpr int kGraphSteps = 20;   // Adam steps captured per search graph (see felix_search)
struct Chunks {
  const CostModel* cm = nullptr;
  uint64_t cm_uid = 0;
  int64_t n = -1;
  int K = 0;
  std::vector<int64_t> off, cnt;
  std::vector<std::unique_ptr<Plan>> plans;
  std::vector<cudaStream_t> streams;       // capture-time branch streams / per-chunk launch streams
  cudaGraphExec_t graph = nullptr;            // kGraphSteps Adam steps per launch
  cudaGraphExec_t graph_tail = nullptr;       // the remainder (n_steps % kGraphSteps steps)
  int graph_tail_steps = 0;
  std::vector<double> graph_key;
  std::vector<cudaGraphExec_t> chunk_graphs;   // independent per-chunk step graphs (no per-step join)
  std::vector<double> chunk_key;
  cudaEvent_t ev_fork = nullptr;
  std::vector<cudaEvent_t> ev_join;
  ~Chunks() {
    if (graph) cudaGraphExecDestroy(graph);
    if (graph_tail) cudaGraphExecDestroy(graph_tail);
    for (auto g : chunk_graphs) if (g) cudaGraphExecDestroy(g);
    if (ev_fork) cudaEventDestroy(ev_fork);
    for (auto e : ev_join) cudaEventDestroy(e);
    for (auto st : streams) cudaStreamDestroy(st);
  }
};

struct ProfEvent { int cls; cudaEvent_t a, b; };

// felix_search_group workspace: one MLP plan over the rows of every member space; per member its Adam
// state and step counter; a one-step graph (fork: DAG forwards, join: MLP, fork: reverse/Adam, join)
struct GroupCache {
  uint64_t cm_uid = 0;
  std::vector<uint64_t> space_uid;   // member identities (uid + statement count), never raw addresses
  std::vector<int> space_ns;
  std::vector<int64_t> n, row_off;
  std::unique_ptr<Plan> plan;
  std::vector<std::unique_ptr<DevBuf>> m, v, step_ctr;
  std::vector<std::unique_ptr<DevBuf>> sc_part, sc_pen;   // split-cone buffers per member (see Plan)
  std::vector<cudaStream_t> streams;
  cudaGraphExec_t graph = nullptr;            // graph_steps Adam steps per launch (see felix_search)
  cudaGraphExec_t graph_tail = nullptr;
  int graph_tail_steps = 0;
  std::vector<double> key;
  ~GroupCache() {
    if (graph) cudaGraphExecDestroy(graph);
    if (graph_tail) cudaGraphExecDestroy(graph_tail);
    for (auto st : streams) cudaStreamDestroy(st);
  }
};

}  // namespace felix

static constexpr int kModuleParts = 8;   // kernels of a generated module (codegen.cpp FELIX_PART)

struct felix_space {
  uint64_t uid = felix::next_uid();   // identity for workspace caches (see GroupCache)
  int device = 0;
  felix::SpaceDesc desc;
  felix::RoundTables rt;
  int K0p = 96;
  // device copies of the rounding tables
  felix::DevBuf d_comp_nvars, d_comp_var0, d_comp_vars, d_comp_eoff, d_comp_tcount, d_tuples, d_lnf;
  felix::DevBuf d_int_vars, d_int_lo, d_int_cnt, d_int_toff, d_int_thr;
  felix::DevBuf d_comp_ns, d_comp_s0, d_comp_sext, d_var_smask, d_var_doff, d_var_dcnt, d_dval, d_dln, d_bnb_sel, d_all_sel;
  // NVRTC modules, one per cone-partition width P (compiled on first use)
  struct Module {
    cudaLibrary_t libs[kModuleParts] = {};   // one library per generated kernel (compiled in parallel)
    cudaKernel_t f_fwd = nullptr, f_rev_adam = nullptr, f_rev_eval = nullptr, f_hard = nullptr, f_init = nullptr;
    cudaKernel_t f_rev_sc = nullptr, f_fwd_adam = nullptr, f_adam_sc = nullptr;   // split-cone search kernels
    int P = 1, R = 1, rev_smem = 0, regs_fwd = 0, regs_rev = 0;   // cone groups, replicas per block
    std::string source;
  };
  std::map<int, Module> modules;
  double nvrtc_ms = 0;
  int regs_fwd = 0, regs_rev = 0;
  int64_t flops_fwd = 0, flops_rev = 0;
  // workspace caches (search: chunked; eval: one chunk) + scratch
  std::unique_ptr<felix::Chunks> search_chunks, eval_chunks;
  std::unique_ptr<felix::GroupCache> group_cache;   // felix_search_group with this space first
  felix::DevBuf sched, valid, phi64, score, act64a, act64b, alive, rec_cand, rec_cnt, fin_cand, fin_cnt, o_idx, o_score, o_sched;
  felix::DevBuf o_pack;
  felix::DevBuf rec_cand2, rec_cnt2;         // multi-phase top-k: records of the odd phases                       // felix_round_topk outputs, one contiguous block: [count | idx | score | sched]
  void* h_pack = nullptr;                     // pinned host copy of o_pack (one D2H copy per call)
  size_t h_pack_bytes = 0;
  // varValuesHistory (Alg. 1 l.13/17) of the last search run with history != 0: per-step rounded points,
  // each seed's previous schedule, the schedule hash set and the pool of distinct schedules
  felix::DevBuf h_sched, h_last, h_slot_h, h_slot_i, h_pool_sched, h_pool_key, h_cnt, o_step;   // h_cnt: count, overflow
  bool h_valid = false;
  int64_t h_n = 0, h_cap = 0, h_index_base = 0;
  uint64_t h_mask = 0;
  // profiling
  bool profiling = false;
  std::vector<felix::ProfEvent> prof;
  double prof_ms[4] = {0, 0, 0, 0};
  int64_t prof_launches[4] = {0, 0, 0, 0};
  ~felix_space() {
    if (h_pack) cudaFreeHost(h_pack);
    for (auto& e : prof) { cudaEventDestroy(e.a); cudaEventDestroy(e.b); }
    for (auto& kv : modules)
      for (cudaLibrary_t l : kv.second.libs) if (l) cudaLibraryUnload(l);
  }
};

struct felix_costmodel : felix::CostModel {};

namespace felix {

// ============================================================================ helpers
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    CUDA_OK(cudaGetDevice(&prev));
    if (prev != dev) CUDA_OK(cudaSetDevice(dev));
    CUDA_OK(cudaFree(nullptr));   // ensure the primary context exists (driver API shares it)
  }
  ~DeviceGuard() { if (prev >= 0) cudaSetDevice(prev); }
};

static void check_device(int dev) {
  int count = 0;
  if (cudaGetDeviceCount(&count) != cudaSuccess || count == 0)
    FELIX_THROW(FELIX_E_CUDA, "no CUDA device available (libfelix has no CPU fallback)");
  if (dev < 0 || dev >= count) FELIX_THROW(FELIX_E_INVALID_ARG, "device index out of range");
  cudaDeviceProp p{};
  CUDA_OK(cudaGetDeviceProperties(&p, dev));
  if (p.major != 10) FELIX_THROW(FELIX_E_CUDA, std::string("libfelix is built for sm_100a; device is ") + p.name);
}

template <class T>
static void upload(DevBuf& d, const std::vector<T>& h) {
  d.alloc(std::max<size_t>(h.size() * sizeof(T), 16));
  if (!h.empty()) CUDA_OK(cudaMemcpy(d.p, h.data(), h.size() * sizeof(T), cudaMemcpyHostToDevice));
}

static void ensure(DevBuf& d, size_t bytes) {
  if (d.bytes < bytes) d.alloc(bytes);
}

static int arity(int op) {
  switch (op) {
    case FELIX_OP_CONST: case FELIX_OP_VAR: return 0;
    case FELIX_OP_NEG: case FELIX_OP_EXP: case FELIX_OP_LOG: case FELIX_OP_SQRT: case FELIX_OP_NOT: case FELIX_OP_POW: return 1;
    case FELIX_OP_SELECT: return 3;
    default: return 2;
  }
}
static bool is_bool_op(int op) {
  return op == FELIX_OP_GT || op == FELIX_OP_GE || op == FELIX_OP_LT || op == FELIX_OP_LE || op == FELIX_OP_EQ ||
         op == FELIX_OP_NE || op == FELIX_OP_AND || op == FELIX_OP_OR || op == FELIX_OP_NOT;
}

// ============================================================================ rounding tables
static std::vector<int64_t> divisors(int64_t n) {
  std::vector<int64_t> d;
  for (int64_t k = 1; k * k <= n; ++k)
    if (n % k == 0) { d.push_back(k); if (k * k != n) d.push_back(n / k); }
  std::sort(d.begin(), d.end());
  return d;
}

void build_round_tables(const SpaceDesc& d, RoundTables& t) {
  const int M = d.n_vars;
  std::vector<int> parent(M);
  std::iota(parent.begin(), parent.end(), 0);
  std::function<int(int)> find = [&](int j) { while (parent[j] != j) { parent[j] = parent[parent[j]]; j = parent[j]; } return j; };
  for (auto& sv : d.split_vars) for (size_t k = 1; k < sv.size(); ++k) parent[find(sv[k])] = find(sv[0]);
  std::vector<std::vector<int>> comps;
  std::vector<int> root_of(M, -1);
  for (int j = 0; j < M; ++j) {
    if (d.vars[j].kind != FELIX_VAR_SPLIT) continue;
    int r = find(j);
    if (root_of[r] < 0) { root_of[r] = (int)comps.size(); comps.push_back({}); }
    comps[root_of[r]].push_back(j);
  }
  for (auto& comp : comps) {
    if (comp.size() > 8) FELIX_THROW(FELIX_E_UNSUPPORTED, "split component with more than 8 variables");
    std::vector<int> sp;   // splits touching the component
    for (size_t s = 0; s < d.split_vars.size(); ++s)
      for (int v : d.split_vars[s]) if (std::find(comp.begin(), comp.end(), v) != comp.end()) { sp.push_back((int)s); break; }
    if (sp.size() > static_cast<size_t>(kRoundMaxSplits))
      FELIX_THROW(FELIX_E_UNSUPPORTED, "split component touching more than 16 splits");
    auto in_split = [&](int q, int j) {
      return std::find(d.split_vars[sp[q]].begin(), d.split_vars[sp[q]].end(), j) != d.split_vars[sp[q]].end();
    };
    const int nv = (int)comp.size();
    const int ci = (int)t.comp_nvars.size();
    t.comp_nvars.push_back(nv);
    t.comp_var0.push_back((int)t.comp_vars.size());
    for (int j : comp) t.comp_vars.push_back(j);
    // branch-and-bound data (always built: felix_tune("round_bnb", 1) searches every component that way)
    t.comp_ns.push_back((int)sp.size());
    t.comp_s0.push_back((int)t.comp_sext.size());
    for (int q : sp) t.comp_sext.push_back(d.split_extent[q]);
    for (int j : comp) {
      uint32_t mask = 0;
      int64_t g = 0;
      for (size_t q = 0; q < sp.size(); ++q)
        if (in_split((int)q, j)) { mask |= 1u << q; g = std::gcd(g, d.split_extent[sp[q]]); }
      t.var_smask.push_back(mask);
      t.var_doff.push_back((int64_t)t.dval.size());
      const auto dv = divisors(g);
      t.var_dcnt.push_back((int32_t)dv.size());
      for (int64_t x : dv) { t.dval.push_back(x); t.dln.push_back(std::log((double)x)); }
    }
    // the tuple table, in lexicographic order, unless it exceeds kRoundTableMax rows
    t.comp_toff.push_back(t.n_tuples_total);
    t.comp_eoff.push_back((int64_t)t.tuples.size());
    const size_t tup0 = t.tuples.size();
    int64_t count = 0;
    bool overflow = false;
    std::vector<int64_t> rem(sp.size());
    for (size_t q = 0; q < sp.size(); ++q) rem[q] = d.split_extent[sp[q]];
    std::vector<int32_t> cur(nv);
    std::function<void(int)> rec = [&](int k) {
      if (overflow) return;
      if (k == nv) {
        if (++count > kRoundTableMax) { overflow = true; return; }
        for (int q = 0; q < nv; ++q) { t.tuples.push_back(cur[q]); t.lnf.push_back(std::log((double)cur[q])); }
        return;
      }
      const int j = comp[k];
      int64_t g = 0;
      for (size_t q = 0; q < sp.size(); ++q)
        if (in_split((int)q, j)) g = std::gcd(g, rem[q]);
      for (int64_t dv : divisors(g)) {
        if (overflow) return;
        std::vector<int64_t> save = rem;
        for (size_t q = 0; q < sp.size(); ++q)
          if (in_split((int)q, j)) rem[q] /= dv;
        cur[k] = (int32_t)dv;
        rec(k + 1);
        rem = save;
      }
    };
    rec(0);
    if (overflow) {
      t.tuples.resize(tup0);
      t.lnf.resize(tup0);
      t.comp_tcount.push_back(-1);
      t.bnb_comps.push_back(ci);
    } else {
      t.comp_tcount.push_back(count);
      t.n_tuples_total += count;
    }
  }
  for (int j = 0; j < M; ++j) {
    if (d.vars[j].kind != FELIX_VAR_INT) continue;
    t.int_vars.push_back(j);
    t.int_lo.push_back(d.vars[j].lo);
    t.int_hi.push_back(d.vars[j].hi);
    t.int_toff.push_back((int64_t)t.int_thr.size());
    for (int64_t k = d.vars[j].lo; k < d.vars[j].hi; ++k) t.int_thr.push_back(std::log((double)k + 0.5));
  }
}

// ============================================================================ NVRTC
static std::vector<char> nvrtc_compile(const std::string& source, int part = 0) {
  nvrtcProgram prog;
  if (nvrtcCreateProgram(&prog, source.c_str(), "felix_space.cu", 0, nullptr, nullptr) != NVRTC_SUCCESS)
    FELIX_THROW(FELIX_E_NVRTC, "nvrtcCreateProgram failed");
  const std::string def = "-DFELIX_PART=" + std::to_string(part);
  const char* opts[] = {"--gpu-architecture=sm_100a", "-std=c++17", "-lineinfo", "--fmad=true", def.c_str()};
  nvrtcResult rc = nvrtcCompileProgram(prog, part > 0 ? 5 : 4, opts);
  if (rc != NVRTC_SUCCESS) {
    size_t ls = 0;
    nvrtcGetProgramLogSize(prog, &ls);
    std::string log(ls, '\0');
    nvrtcGetProgramLog(prog, &log[0]);
    nvrtcDestroyProgram(&prog);
    FELIX_THROW(FELIX_E_NVRTC, "NVRTC compile failed: " + log.substr(0, 4000));
  }
  size_t cs = 0;
  nvrtcGetCUBINSize(prog, &cs);
  std::vector<char> cubin(cs);
  nvrtcGetCUBIN(prog, cubin.data());
  nvrtcDestroyProgram(&prog);
  return cubin;
}

// The generated module's kernels, one NVRTC program each (codegen.cpp guards every kernel with
// FELIX_PART == k): the eight compile on parallel host threads, ~3x faster than one program at C2
// (7.5 s -> 2.7 s on 8 cores), and ptxas sees one kernel's straight-line code at a time.
static const char* const kModuleKernels[kModuleParts] = {"felix_fwd", "felix_fwd_adam", "felix_rev_adam", "felix_rev_eval",
                                                          "felix_rev_sc", "felix_adam_sc", "felix_hard", "felix_init"};

// Process-wide cubin cache keyed by the generated source: spaces with the same expression DAG and
// launch shape (a re-created space, the same subgraph in another task list) load the compiled kernels
// instead of recompiling them.  Bounded; cleared wholesale when full.
static std::mutex g_cubin_mu;
static std::map<std::string, std::shared_ptr<const std::vector<std::vector<char>>>> g_cubins;

static std::shared_ptr<const std::vector<std::vector<char>>> compile_module_parts(const std::string& source) {
  {
    std::lock_guard<std::mutex> lk(g_cubin_mu);
    auto it = g_cubins.find(source);
    if (it != g_cubins.end()) return it->second;
  }
  auto parts = std::make_shared<std::vector<std::vector<char>>>(kModuleParts);
  std::vector<std::string> err(kModuleParts);
  std::atomic<int> next{0};
  auto worker = [&]() {
    for (int k; (k = next.fetch_add(1)) < kModuleParts;) {
      try { (*parts)[k] = nvrtc_compile(source, k + 1); } catch (const std::exception& e) { err[k] = e.what(); }
    }
  };
  const int nt = std::max(1, std::min<int>(kModuleParts, static_cast<int>(std::thread::hardware_concurrency())));
  std::vector<std::thread> th;
  for (int t = 1; t < nt; ++t) th.emplace_back(worker);
  worker();
  for (auto& t : th) t.join();
  for (int k = 0; k < kModuleParts; ++k)
    if (!err[k].empty()) FELIX_THROW(FELIX_E_NVRTC, std::string(kModuleKernels[k]) + ": " + err[k]);
  std::lock_guard<std::mutex> lk(g_cubin_mu);
  if (g_cubins.size() >= 64) g_cubins.clear();
  g_cubins.emplace(source, parts);
  return parts;
}

static felix_space::Module& get_module(felix_space* s, int P, int R = 1, int dphi_parts = 1) {
  // the forward kernel stages NREP x NS x 32 x (K0P+1) floats + NREP x NV x 32 doubles statically
  if (R > 1 && static_cast<int64_t>(R) * (s->desc.n_statements * 32 * (s->K0p + 1) * 4 + s->desc.n_vars * 32 * (8 + 4) + 64) > 48 * 1024)
    R = 1;
  const bool trace = g_tune.trace.load() != 0;
  const int key = P + 64 * R + (trace ? 4096 : 0) + 8192 * dphi_parts;
  auto it = s->modules.find(key);
  if (it != s->modules.end()) return it->second;
  felix_space::Module mod;
  mod.P = P;
  mod.R = R;
  CodegenInfo info;
  mod.source = generate_dag_module(s->desc, s->K0p, P, R, trace, dphi_parts, &info);
  s->flops_fwd = info.flops_fwd;
  s->flops_rev = info.flops_rev;
  mod.rev_smem = info.rev_smem_bytes;
  auto t0 = std::chrono::steady_clock::now();
  const auto cubins = compile_module_parts(mod.source);
  cudaKernel_t* slots[kModuleParts] = {&mod.f_fwd, &mod.f_fwd_adam, &mod.f_rev_adam, &mod.f_rev_eval,
                                       &mod.f_rev_sc, &mod.f_adam_sc, &mod.f_hard, &mod.f_init};
  for (int k = 0; k < kModuleParts; ++k) {
    CUDA_OK(cudaLibraryLoadData(&mod.libs[k], (*cubins)[k].data(), nullptr, nullptr, 0, nullptr, nullptr, 0));
    CUDA_OK(cudaLibraryGetKernel(slots[k], mod.libs[k], kModuleKernels[k]));
  }
  for (cudaKernel_t k : {mod.f_rev_adam, mod.f_rev_eval})
    CUDA_OK(cudaFuncSetAttribute(reinterpret_cast<const void*>(k), cudaFuncAttributeMaxDynamicSharedMemorySize, mod.rev_smem));
  cudaFuncAttributes fa{};
  CUDA_OK(cudaFuncGetAttributes(&fa, reinterpret_cast<const void*>(mod.f_fwd)));
  mod.regs_fwd = fa.numRegs;
  CUDA_OK(cudaFuncGetAttributes(&fa, reinterpret_cast<const void*>(mod.f_rev_adam)));
  mod.regs_rev = fa.numRegs;
  s->nvrtc_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  s->regs_fwd = mod.regs_fwd;
  s->regs_rev = mod.regs_rev;
  return s->modules.emplace(key, std::move(mod)).first->second;
}

// Replicas of the cone groups per block (cone-group kernels): warps running the same cone's straight-line
// code share the SM's instruction fetches.  Measured at C2: R=2 takes the reverse kernel from 16.9 to
// 15.3 us but the step only +0.6 %; R=4 exceeds the static shared budget.  Default 1; felix_tune overrides.
static int choose_R(int64_t n, int P) {
  (void)n; (void)P;
  const int r = g_tune.R.load();
  return (r == 1 || r == 2 || r == 4) ? r : 1;
}

// Cone-partition width: enough warps to give every SM ~8 resident warps of expression work.
static int choose_P(int64_t n) {
  const int p = g_tune.P.load();
  if (p == 1 || p == 2 || p == 4 || p == 8 || p == 16) return p;
  // measured on B200 (C2 space, per-class event timing): P=4 best at 4096 candidates, P=2 at 32768,
  // P=1 once the population alone fills the SMs
  int P = 1;
  if (n <= 8192) P = 4;
  else if (n <= 65536) P = 2;
  return P;
}

// Launch helpers.  Search kernels: CTA = P warps x 32 candidates (cone partition); hard / sampler
// kernels: one candidate per thread, 128-thread CTAs.
static void launch_cfg(const void* f, dim3 grid, dim3 block, size_t smem, void** args, cudaStream_t st, bool pdl) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  if (pdl && pdl_mask()) { cfg.attrs = &g_pdl_attr; cfg.numAttrs = 1; }
  CUDA_OK(cudaLaunchKernelExC(&cfg, f, args));
}
static void launch_grouped(cudaKernel_t f, int P, int R, int64_t n, size_t smem, void** args, cudaStream_t st, bool pdl) {
  if (n <= 0) return;
  launch_cfg(reinterpret_cast<const void*>(f), dim3(static_cast<unsigned>((n + 32 * R - 1) / (32 * R))), dim3(32 * P * R),
             smem, args, st, pdl);
}
// felix_init: one warp per candidate (32 rejection attempts in flight)
static void launch_warp_per_item(cudaKernel_t f, int64_t n, void** args, cudaStream_t st) {
  if (n <= 0) return;
  launch_cfg(reinterpret_cast<const void*>(f), dim3(static_cast<unsigned>((n * 32 + 127) / 128)), dim3(128), 0, args, st, false);
}
static void launch_flat(cudaKernel_t f, int64_t n, void** args, cudaStream_t st) {
  if (n <= 0) return;
  launch_cfg(reinterpret_cast<const void*>(f), dim3(static_cast<unsigned>((n + 127) / 128)), dim3(128), 0, args, st, false);
}

// Split-cone reverse kernel (codegen.cpp felix_rev_sc): one cone per CTA for W x 32 candidates, partial
// adjoints through global memory; the next step's forward (felix_fwd_adam) sums them and applies Adam,
// felix_adam_sc after the last step.  Default for single-space searches; felix_tune("split_cone", 0)
// selects felix_rev_adam, 1 forces it in group searches too (measured there with an earlier variant:
// C3 1.66e8 -> 1.65e8, C4 2.25e8 -> 2.08e8 cand-steps/s, so groups keep felix_rev_adam by default).
// Not with history rounding (it rounds the caller's y before each step's forward, i.e. before Adam).
static bool use_sc(bool group = false, int64_t min_member_n = 0) {
  const int v = g_tune.sc.load();
  if (v == 0) return false;
  if (v == 1) return true;
  // groups: split-cone once every member has >= 2048 candidates (measured, FP32 reverse: C4 shards of
  // 2048 / 4096 seeds per task +7 % / +13 %, C3 with 1024 per task -8 %)
  return !group || min_member_n >= 2048;
}
__global__ void set_int_kernel(int* p, int v) { *p = v; }
// Split-cone searches: at least two cones (measured at the C5 shard, 131072 candidates: 2.53e8 at P = 1,
// 2.72e8 at P = 2 cand-steps/s) and two replicas of the cone groups per felix_fwd_adam block (warps on the
// same cone share instruction fetches; C2 forward 14.8 -> 12.8 us).  felix_tune overrides.
static int choose_P_sc(int P) { return (P == 1 && g_tune.P.load() < 0) ? 2 : P; }
static int choose_R_sc() {
  const int r = g_tune.R.load();
  return (r == 1 || r == 2 || r == 4) ? r : 2;
}
// warps per split-cone CTA: about one CTA per SM (felix_tune("sc_warps") overrides).  Measured at C2
// (P = 4, 128 candidate groups) without PDL edges (profiles/r02/sc_warps_nopdl.log): W = 4 (128 CTAs)
// 9.13e7 cand-steps/s, W = 8 9.04e7, W = 6 9.03e7, W = 2 8.95e7.  (With PDL edges W = 2 had measured
// best, profiles/r02/sc_warps.log: the early-resident next kernel then competed with fewer, larger CTAs.)
static int choose_scw(int64_t n, int P) {
  const int w0 = g_tune.scw.load();
  if (w0 >= 1 && w0 <= 8) return w0;
  const int64_t groups = (n + 31) / 32;
  int64_t w = (groups * P + 147) / 148;
  return static_cast<int>(std::max<int64_t>(1, std::min<int64_t>(8, w)));
}
static int64_t sc_groups(int64_t n, int W) { return ((n + 31) / 32 + W - 1) / W; }
static void launch_sc(cudaKernel_t f, int P, int W, int64_t n, void** args, cudaStream_t st, bool pdl) {
  if (n <= 0) return;
  launch_cfg(reinterpret_cast<const void*>(f), dim3(static_cast<unsigned>(sc_groups(n, W) * P)), dim3(32 * W),
             0, args, st, pdl);
}

// ============================================================================ plan
static int choose_bn(int64_t m_tiles, int N) {
  // prefer >= one full wave of CTAs (148 SMs) before larger tiles
  if (N % 128 == 0 && m_tiles * (N / 128) >= 2 * 148) return 128;
  if (N % 64 == 0) return 64;
  FELIX_THROW(FELIX_E_UNSUPPORTED, "hidden dim must be a multiple of 64");
}

// MLP workspace for n MLP rows (and Adam state for n_vars x n_cand when n_cand > 0)
static std::unique_ptr<Plan> build_plan_rows(int device, const CostModel* cm, int64_t n, int n_vars, int64_t n_cand) {
  auto p = std::make_unique<Plan>();
  p->cm = cm;
  p->n = n;
  // 2-SM chain pairs: rows padded to whole 256-row pairs (the OOB rows are zero-filled by TMA and
  // clipped on store; every row-block flag exists)
  p->chain_cg = g_tune.chain_cg.load() == 2 ? 2 : 1;
  p->n_pad = (n + 128 * p->chain_cg - 1) / (128 * p->chain_cg) * (128 * p->chain_cg);
  const int L = cm->n_layers;
  const auto& d = cm->dims;
  const int64_t np = p->n_pad;
  const int K0p = cm->K0p;
  p->phi_hi.alloc(np * K0p * 2);
  p->phi_lo.alloc(np * K0p * 2);
  p->act_hi.resize(L);
  p->act_lo.resize(L);
  p->mask.resize(L);
  for (int l = 1; l <= L - 1; ++l) {
    p->act_hi[l] = std::make_unique<DevBuf>();
    p->act_lo[l] = std::make_unique<DevBuf>();
    p->act_hi[l]->alloc(np * d[l] * 2);
    p->act_lo[l]->alloc(np * d[l] * 2);
    if (l <= L - 2) {
      p->mask[l] = std::make_unique<DevBuf>();
      p->mask[l]->alloc(np * (d[l] / 32) * 4);
    }
  }
  // split-K of the chain's dL/dphi layer (K = d1): ksplit contiguous K ranges on ksplit CTAs per row block,
  // each writing a partial slab (measured at C2: see DESIGN.md §8); only while every part fits one wave
  int sms0 = 148;
  CUDA_OK(cudaDeviceGetAttribute(&sms0, cudaDevAttrMultiProcessorCount, device));
  int dphi_split = 1;
  {
    const int nkb1 = (d[1] + GEMM_BK - 1) / GEMM_BK;
    const int ks = g_tune.dphi_ksplit.load();
    auto fits = [&](int sp) { return nkb1 % sp == 0 && (np / 128) * sp <= sms0; };
    if ((ks == 2 || ks == 4) && nkb1 % ks == 0) dphi_split = ks;
    else if (ks < 0 && fits(4)) dphi_split = 4;
  }
  p->dphi.alloc(static_cast<size_t>(dphi_split) * K0p * np * 4);
  p->m.alloc(static_cast<size_t>(n_vars) * n_cand * 4);
  p->v.alloc(static_cast<size_t>(n_vars) * n_cand * 4);
  p->step_ctr.alloc(16);
  const int64_t mt = np / 128;
  // forward GEMMs, layer l = 1..L-1 (W index l-1)
  for (int l = 1; l <= L - 1; ++l) {
    GemmLaunch g;
    const bool head = (l == L - 1);
    g.epi = head ? EPI_HEAD : EPI_RELU;
    const int N = d[l], Kdim = (l == 1) ? K0p : d[l - 1];
    g.bn = choose_bn(mt, N);
    const void* a_hi = (l == 1) ? p->phi_hi.p : p->act_hi[l - 1]->p;
    const void* a_lo = (l == 1) ? p->phi_lo.p : p->act_lo[l - 1]->p;
    g.a_hi = make_tmap(a_hi, n, Kdim, 128);
    g.a_lo = make_tmap(a_lo, n, Kdim, 128);
    g.w_hi = cm->W_hi[l - 1]->p;
    g.w_lo = cm->W_lo[l - 1]->p;
    g.b_hi = make_tmap(g.w_hi, N, Kdim, g.bn);
    g.b_lo = make_tmap(g.w_lo, N, Kdim, g.bn);
    g.c_hi = make_tmap(p->act_hi[l]->p, n, N, 128);
    g.c_lo = make_tmap(p->act_lo[l]->p, n, N, 128);
    GemmArgs& a = g.args;
    a.M = static_cast<int>(n); a.N = N; a.K = Kdim;
    a.bias = cm->bias[l - 1]->as<float>();
    a.out_hi = p->act_hi[l]->as<__half>();
    a.out_lo = p->act_lo[l]->as<__half>();
    a.ld_out = N;
    if (head) {
      a.head_w = cm->head_w.as<float>();
      p->n_head_tiles = N / g.bn;
      p->c_part.alloc(static_cast<size_t>(N / 16) * np * 4);      // room for any partial width >= 16
      a.c_part = p->c_part.as<float>();
      a.ld_c = static_cast<int>(np);
    } else {
      a.mask_out = p->mask[l]->as<uint32_t>();
      a.ld_mask = static_cast<int>(np);
    }
    g.grid = dim3(static_cast<unsigned>(mt), N / g.bn);
    g.stages = std::min(gemm_max_stages(g.bn), (Kdim + GEMM_BK - 1) / GEMM_BK);
    p->gemms.push_back(g);
  }
  // backward GEMMs: delta_{l-1} = (delta_l W_l) (.) m_{l-1} for l = L-1..2, then dphi = delta_1 W_1
  for (int l = L - 1; l >= 1; --l) {
    GemmLaunch g;
    const bool last = (l == 1);
    const int N = last ? K0p : d[l - 1], Kdim = d[l];
    g.epi = last ? EPI_F32T : EPI_MASK;
    g.bn = last ? K0p : choose_bn(mt, N);
    g.a_hi = make_tmap(p->act_hi[l]->p, n, Kdim, 128);
    g.a_lo = make_tmap(p->act_lo[l]->p, n, Kdim, 128);
    g.w_hi = cm->WT_hi[l - 1]->p;
    g.w_lo = cm->WT_lo[l - 1]->p;
    g.b_hi = make_tmap(g.w_hi, N, Kdim, g.bn);
    g.b_lo = make_tmap(g.w_lo, N, Kdim, g.bn);
    GemmArgs& a = g.args;
    a.M = static_cast<int>(n); a.N = N; a.K = Kdim;
    g.c_hi = last ? g.a_hi : make_tmap(p->act_hi[l - 1]->p, n, N, 128);
    g.c_lo = last ? g.a_lo : make_tmap(p->act_lo[l - 1]->p, n, N, 128);
    if (last) {
      a.out_f32 = p->dphi.as<float>();
      a.ld_f32 = static_cast<int>(np);
      a.n_valid = d[0];
    } else {
      a.out_hi = p->act_hi[l - 1]->as<__half>();
      a.out_lo = p->act_lo[l - 1]->as<__half>();
      a.ld_out = N;
      a.mask_in = p->mask[l - 1]->as<uint32_t>();
      a.ld_mask = static_cast<int>(np);
    }
    g.grid = dim3(static_cast<unsigned>(mt), N / g.bn);
    g.stages = std::min(gemm_max_stages(g.bn), (Kdim + GEMM_BK - 1) / GEMM_BK);
    p->gemms.push_back(g);
  }
  // persistent chain: same layers, BN <= 128, one CTA per SM
  int sms = 148;
  CUDA_OK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device));
  if (static_cast<int>(p->gemms.size()) > CHAIN_MAX_LAYERS) FELIX_THROW(FELIX_E_UNSUPPORTED, "too many MLP layers");
  p->chain.n_layers = static_cast<int>(p->gemms.size());
  p->chain.m_tiles = static_cast<int>(mt);
  p->grid_bar.alloc(64);
  CUDA_OK(cudaMemset(p->grid_bar.p, 0, 64));
  p->chain.grid_bar = p->grid_bar.as<unsigned int>();
  int max_tiles = 1;
  for (size_t i = 0; i < p->gemms.size(); ++i) {
    const GemmLaunch& g = p->gemms[i];
    ChainLayer& L = p->chain.layer[i];
    L.args = g.args;
    L.epi = g.epi;
    const int N = g.args.N;
    int bn = g.bn;
    L.ksplit = 1;
    if (g.epi == EPI_F32T) {
      // dL/dphi (K = d1 = 512, N = K0p): its A row block is the largest operand a CTA ingests, and with
      // one N tile only mt CTAs work: split K over dphi_split CTAs (partial slabs), else 32-wide N tiles
      // spread it over 3x the CTAs while they fit in one wave
      bn = g.bn;                                                          // K0p (<= 128 required)
      if (dphi_split > 1) L.ksplit = dphi_split;
      else if (N % 32 == 0 && mt * (N / 32) <= sms) bn = 32;
    }
    else bn = (N % 128 == 0 && mt * (N / 128) >= sms * 2 / 3) ? 128 : 64;
    if (bn > CHAIN_BN_MAX) FELIX_THROW(FELIX_E_UNSUPPORTED, "chain tile N > 128");
    L.bn = bn;
    L.n_tiles_n = N / bn;
    L.f32t_tma = 0;
    if (g.epi == EPI_F32T && bn <= CHAIN_BN_MAX && g_tune.dphi_tma.load() != 0) {
      // the dL/dphi slabs [ksplit * N][n_pad] fp32 through one TMA store per tile (mlp_chain.cuh)
      L.c_f32 = make_tmap_f32(g.args.out_f32, static_cast<int64_t>(L.ksplit) * N, g.args.ld_f32, GEMM_BM, bn);
      L.f32t_tma = 1;
    }
    L.n_tiles = static_cast<int>(mt) * L.n_tiles_n;
    const int ccg = p->chain_cg;
    L.idesc = ptx::idesc_f16_f32(GEMM_BM * ccg, static_cast<uint32_t>(bn));
    L.idesc_cat = ptx::idesc_f16_f32(GEMM_BM, static_cast<uint32_t>(2 * bn));   // [B_hi ; B_lo] (FELIX_CHAIN_NCAT, CG = 1)
    L.a_hi = g.a_hi; L.a_lo = g.a_lo; L.c_hi = g.c_hi; L.c_lo = g.c_lo;
    L.b_hi = make_tmap(g.w_hi, N, g.args.K, bn / ccg);     // CG = 2: each CTA loads half of the tile's weight rows
    L.b_lo = make_tmap(g.w_lo, N, g.args.K, bn / ccg);
    // the first backward layer takes the 0/1 mask of the head layer as its A operand and the head row
    // folded into its weights (exact A: no A lo loads, one N-concatenated MMA per K step)
    L.a_exact = 0;
    L.head_exact = 0;
    if (i == static_cast<size_t>(cm->n_layers - 1) && i > 0 && p->gemms[i - 1].epi == EPI_HEAD) {
      L.a_exact = 1;
      p->chain.layer[i - 1].head_exact = 1;
      L.b_hi = make_tmap(cm->WTs_hi.p, N, g.args.K, bn / ccg);
      L.b_lo = make_tmap(cm->WTs_lo.p, N, g.args.K, bn / ccg);
    }
    if (g.epi == EPI_HEAD && use_chain()) p->n_head_tiles = CHAIN_EPI_NQ * (N / bn);   // chain: one partial per column slice
    max_tiles = std::max(max_tiles, static_cast<int>((mt + ccg - 1) / ccg) * L.n_tiles_n * L.ksplit * ccg);   // CTAs the layer can use
  }
  p->chain_grid = std::min(sms / p->chain_cg * p->chain_cg, max_tiles);
  // Grid chain with per-row-block dataflow flags (cooperative launch: every CTA resident): at C2 44.2 us
  // per Adam step vs 45.7 us for a cluster chain (one 4-CTA cluster per row block, cluster barriers; removed)
  // and faster above 37 row blocks (n=8192: 56 vs 90 us).  The epoch is the step counter the forward DAG
  // kernel bumps before every chain launch.
  p->chain_flags.alloc(static_cast<size_t>(p->chain.n_layers) * mt * CHAIN_FLAG_STRIDE * 4);
  CUDA_OK(cudaMemset(p->chain_flags.p, 0, p->chain_flags.bytes));
  {
    p->chain.flags = p->chain_flags.as<unsigned int>();
    p->chain.epoch = p->step_ctr.as<int>();
    // own-chunk reuse (mlp_chain.cuh ChainLayer::reuse) where every CTA keeps its row block between two layers
    const bool reuse_ok = CHAIN_EPI_BUFS == 2;
    for (int i = 0; i < p->chain.n_layers; ++i) {
      ChainLayer& Li = p->chain.layer[i];
      Li.reuse = 0;
      if (!reuse_ok || i == 0) continue;
      const ChainLayer& Lp = p->chain.layer[i - 1];
      // every CTA (pair) has at most one tile of each of the two layers and the same N tile in both
      const int64_t units_p = (mt + p->chain_cg - 1) / p->chain_cg * Lp.n_tiles_n, units_i = (mt + p->chain_cg - 1) / p->chain_cg * Li.n_tiles_n;
      const int64_t clusters = p->chain_grid / p->chain_cg;
      if (Lp.epi != EPI_F32T && Li.ksplit == 1 && units_p <= clusters && units_i <= clusters &&
          Lp.n_tiles_n == Li.n_tiles_n && Lp.bn % GEMM_BK == 0)
        Li.reuse = 1;
    }
  }
  // tile-local fused MLP: TenSet widths [K0p, 512, 256, 256, 1] only
  p->tile_ok = L == 4 && d[1] == tile::D1 && d[2] == tile::D2 && d[3] == tile::D3 && K0p <= 128 && K0p % 32 == 0;   // K0p/2 rows: multiple of 16
  if (p->tile_ok) {
    p->tile_cg = g_tune.tile_cg.load() == 2 ? 2 : 1;
    // measured on B200 (C2 space, default MLP): the chain wins at 64 row blocks (8192 rows: 1.24e8 vs
    // 1.14e8 cand-steps/s), the tile kernel at 128 (16384 rows: 2.09e8 vs 1.66e8) -> tile kernel from
    // ~56 % of a wave of 128-row tiles
    p->tile_full_wave = mt * 16 >= static_cast<int64_t>(sms) * 9;
    const int cg = p->tile_cg;
    TileParams& t = p->tile;
    t.phi_hi = make_tmap(p->phi_hi.p, n, K0p, 128);
    t.phi_lo = make_tmap(p->phi_lo.p, n, K0p, 128);
    t.w1_hi = make_tmap(cm->W_hi[0]->p, d[1], K0p, 128 / cg);
    t.w1_lo = make_tmap(cm->W_lo[0]->p, d[1], K0p, 128 / cg);
    t.w2_hi = make_tmap(cm->W_hi[1]->p, d[2], d[1], 128);
    t.w2_lo = make_tmap(cm->W_lo[1]->p, d[2], d[1], 128);
    t.w3_hi = make_tmap(cm->W_hi[2]->p, d[3], d[2], 128);
    t.w3_lo = make_tmap(cm->W_lo[2]->p, d[3], d[2], 128);
    // B1 on the exact mask with the head row folded into W3^T (as the chain's first backward layer)
    t.d2_exact = 1;
    t.w3t_hi = make_tmap(t.d2_exact ? cm->WTs_hi.p : cm->WT_hi[2]->p, d[2], d[3], 128);
    t.w3t_lo = make_tmap(t.d2_exact ? cm->WTs_lo.p : cm->WT_lo[2]->p, d[2], d[3], 128);
    t.w2t_hi = make_tmap(cm->WT_hi[1]->p, d[1], d[2], 128 / cg);
    t.w2t_lo = make_tmap(cm->WT_lo[1]->p, d[1], d[2], 128 / cg);
    t.w1t_hi = make_tmap(cm->WT_hi[0]->p, K0p, d[1], K0p / cg);
    t.w1t_lo = make_tmap(cm->WT_lo[0]->p, K0p, d[1], K0p / cg);
    t.b1 = cm->bias[0]->as<float>();
    t.b2 = cm->bias[1]->as<float>();
    t.b3 = cm->bias[2]->as<float>();
    t.w4 = cm->head_w.as<float>();
    t.c_part = p->c_part.as<float>();
    t.dphi = p->dphi.as<float>();
    t.ld = static_cast<int>(np);
    t.dphi_tma = g_tune.dphi_tma.load() != 0 ? 1 : 0;
    if (t.dphi_tma) t.dphi_map = make_tmap_f32(p->dphi.p, K0p, np, 128, K0p);
    t.n = static_cast<int>(n);
    t.n_tiles = static_cast<int>(mt);
    t.k0p = K0p;
    t.n_valid = d[0];
    t.idesc_128 = ptx::idesc_f16_f32(128 * cg, 128);
    t.idesc_256 = ptx::idesc_f16_f32(128 * cg, 256);
    t.idesc_k0p = ptx::idesc_f16_f32(128 * cg, static_cast<uint32_t>(K0p));
    const int64_t units = (mt + cg - 1) / cg;
    p->tile_grid = static_cast<int>(std::min<int64_t>(sms / cg, units) * cg);
  }
  p->mode = mlp_mode(*p);
  p->dphi_parts = p->mode == MLP_CHAIN ? dphi_split : 1;   // the tile kernel and the per-layer GEMMs write one slab
  if (p->mode == MLP_TILE) p->n_head_tiles = 2;                           // one partial per column half
  else if (p->mode == MLP_LAYERS) p->n_head_tiles = p->gemms[L - 2].args.N / p->gemms[L - 2].bn;
  return p;
}

static std::unique_ptr<Plan> build_plan(felix_space* s, const CostModel* cm, int64_t n_cand) {
  // the MLP sees one row per (statement, candidate): row = statement * n_cand + candidate
  return build_plan_rows(s->device, cm, n_cand * s->desc.n_statements, s->desc.n_vars, n_cand);
}

// number of concurrent chunks for a population of n (FELIX_CHUNKS overrides; tuned on B200)
static int choose_chunks(int64_t n) {
  const int k = g_tune.chunks.load();
  if (k >= 1 && k <= 16) return k;
  (void)n;   // measured on B200 (C2): 2/4/8 concurrent chunks were 3-14% slower than 1
  return 1;
}

static Chunks& get_chunks(felix_space* s, std::unique_ptr<Chunks>& slot, const CostModel* cm, int64_t n, int K) {
  if (slot && slot->cm_uid == cm->uid && slot->n == n && slot->K == K) return *slot;
  slot.reset();
  auto c = std::make_unique<Chunks>();
  c->cm = cm;
  c->cm_uid = cm->uid;
  c->n = n;
  const int64_t per = ((n + K - 1) / K + 127) / 128 * 128;
  for (int64_t o = 0; o < n; o += per) {
    c->off.push_back(o);
    c->cnt.push_back(std::min(per, n - o));
  }
  c->K = K;
  for (size_t k = 0; k < c->off.size(); ++k) c->plans.push_back(build_plan(s, cm, c->cnt[k]));
  slot = std::move(c);
  return *slot;
}

// ============================================================================ profiling
static void prof_mark(felix_space* s, int cls, cudaStream_t st, bool begin) {
  if (!s->profiling) return;
  if (begin) {
    ProfEvent e{cls, nullptr, nullptr};
    CUDA_OK(cudaEventCreate(&e.a));
    CUDA_OK(cudaEventCreate(&e.b));
    CUDA_OK(cudaEventRecord(e.a, st));
    s->prof.push_back(e);
  } else {
    CUDA_OK(cudaEventRecord(s->prof.back().b, st));
  }
}

// ============================================================================ step pieces
static void run_mlp(felix_space* s, Plan& p, cudaStream_t st);
static void run_forward_mlp(felix_space* s, Plan& p, const felix_space::Module& mod, const float* y, int64_t n,
                            int64_t ldy, cudaStream_t st, int* step_ctr) {
  int ni = static_cast<int>(n), ldi = static_cast<int>(ldy);
  void* phi_hi = p.phi_hi.p;
  void* phi_lo = p.phi_lo.p;
  void* args[] = {&y, &ni, &ldi, &phi_hi, &phi_lo, &step_ctr};
  prof_mark(s, 0, st, true);
  launch_grouped(mod.f_fwd, mod.P, mod.R, n, 0, args, st, true);
  prof_mark(s, 0, st, false);
  s->prof_launches[0] += 1;
  run_mlp(s, p, st);
}

static void run_mlp(felix_space* s, Plan& p, cudaStream_t st) {
  prof_mark(s, 1, st, true);
  const MlpMode mode = static_cast<MlpMode>(p.mode);
  if (mode == MLP_TILE) {
    launch_tile(p, st);
  } else if (mode == MLP_CHAIN) {
    launch_chain(p, st);
  } else {
    for (const auto& g : p.gemms) launch_gemm(g, st);
  }
  prof_mark(s, 1, st, false);
  s->prof_launches[1] += mode == MLP_LAYERS ? static_cast<int64_t>(p.gemms.size()) : 1;
}

}  // namespace felix

using namespace felix;

static std::unique_ptr<felix_space> parse_space(const felix_var* vars, int32_t n_vars, const felix_split* splits,
                                                int32_t n_splits, const felix_node* nodes, int32_t n_nodes,
                                                const int32_t* feature_roots, int32_t n_features,
                                                const int32_t* constraint_roots, int32_t n_constraints) {
  if (n_vars <= 0 || !vars) FELIX_THROW(FELIX_E_INVALID_ARG, "n_vars must be > 0");
  if (n_vars > 64) FELIX_THROW(FELIX_E_UNSUPPORTED, "at most 64 schedule variables");
  if (n_splits < 0 || (n_splits > 0 && !splits)) FELIX_THROW(FELIX_E_INVALID_ARG, "bad splits");
  if (n_nodes <= 0 || !nodes) FELIX_THROW(FELIX_E_INVALID_DAG, "empty DAG");
  if (n_features <= 0 || n_features > 256 || !feature_roots) FELIX_THROW(FELIX_E_SHAPE, "n_features must be in [1, 256]");
  if (n_constraints < 0 || (n_constraints > 0 && !constraint_roots)) FELIX_THROW(FELIX_E_INVALID_ARG, "bad constraints");
  auto s = std::make_unique<felix_space>();
  SpaceDesc& d = s->desc;
  d.n_vars = n_vars;
  d.vars.assign(vars, vars + n_vars);
  std::vector<int> nsplit_of(n_vars, 0);
  for (int j = 0; j < n_vars; ++j) {
    const auto& v = d.vars[j];
    if (v.kind == FELIX_VAR_INT) {
      if (v.lo < 1 || v.hi < v.lo || v.hi > (int64_t(1) << 24)) FELIX_THROW(FELIX_E_INVALID_ARG, "INT var needs 1 <= lo <= hi <= 2^24");
    } else if (v.kind != FELIX_VAR_SPLIT) {
      FELIX_THROW(FELIX_E_INVALID_ARG, "unknown var kind");
    }
  }
  for (int s_ = 0; s_ < n_splits; ++s_) {
    const auto& sp = splits[s_];
    if (sp.extent < 1 || sp.extent >= (int64_t(1) << 31)) FELIX_THROW(FELIX_E_INVALID_ARG, "split extent out of range");
    if (sp.n <= 0 || !sp.vars) FELIX_THROW(FELIX_E_INVALID_ARG, "empty split");
    std::vector<int32_t> sv(sp.vars, sp.vars + sp.n);
    for (int j : sv) {
      if (j < 0 || j >= n_vars) FELIX_THROW(FELIX_E_INVALID_ARG, "split var out of range");
      if (d.vars[j].kind != FELIX_VAR_SPLIT) FELIX_THROW(FELIX_E_INVALID_ARG, "INT var listed in a split");
      nsplit_of[j]++;
    }
    d.split_extent.push_back(sp.extent);
    d.split_vars.push_back(sv);
  }
  for (int j = 0; j < n_vars; ++j)
    if (d.vars[j].kind == FELIX_VAR_SPLIT && nsplit_of[j] == 0) FELIX_THROW(FELIX_E_INVALID_ARG, "SPLIT var in no split");
  // DAG: topological order + types (0 NUM, 1 BOOL, 2 CONST = either)
  d.nodes.assign(nodes, nodes + n_nodes);
  std::vector<int> ty(n_nodes);
  for (int i = 0; i < n_nodes; ++i) {
    const auto& nd = d.nodes[i];
    if (nd.op < 0 || nd.op > FELIX_OP_CEILDIV) FELIX_THROW(FELIX_E_INVALID_DAG, "bad opcode at node " + std::to_string(i));
    const int ar = arity(nd.op);
    const int args[3] = {nd.a, nd.b, nd.c};
    for (int q = 0; q < ar; ++q)
      if (args[q] < 0 || args[q] >= i) FELIX_THROW(FELIX_E_INVALID_DAG, "node " + std::to_string(i) + " argument not an earlier node");
    auto need = [&](int q, int want) {
      const int t = ty[args[q]];
      if (t != 2 && t != want)
        FELIX_THROW(FELIX_E_INVALID_DAG, "type error at node " + std::to_string(i) + (want ? " (expects BOOL)" : " (expects NUM)"));
    };
    if (nd.op == FELIX_OP_VAR) {
      const int j = static_cast<int>(nd.imm);
      if (nd.imm != j || j < 0 || j >= n_vars) FELIX_THROW(FELIX_E_INVALID_DAG, "VAR index out of range");
      ty[i] = 0;
    } else if (nd.op == FELIX_OP_CONST) {
      if (!std::isfinite(nd.imm)) FELIX_THROW(FELIX_E_INVALID_DAG, "non-finite constant");
      ty[i] = 2;
    } else if (nd.op == FELIX_OP_AND || nd.op == FELIX_OP_OR) { need(0, 1); need(1, 1); ty[i] = 1; }
    else if (nd.op == FELIX_OP_NOT) { need(0, 1); ty[i] = 1; }
    else if (nd.op == FELIX_OP_SELECT) { need(0, 1); need(1, 0); need(2, 0); ty[i] = 0; }
    else { for (int q = 0; q < ar; ++q) need(q, 0); ty[i] = is_bool_op(nd.op) ? 1 : 0; }
  }
  for (int k = 0; k < n_features; ++k) {
    const int r = feature_roots[k];
    if (r < 0 || r >= n_nodes || ty[r] == 1) FELIX_THROW(FELIX_E_INVALID_DAG, "feature root must be a NUM node");
    d.froots.push_back(r);
  }
  for (int k = 0; k < n_constraints; ++k) {
    const int r = constraint_roots[k];
    if (r < 0 || r >= n_nodes || ty[r] == 1) FELIX_THROW(FELIX_E_INVALID_DAG, "constraint root must be a NUM node");
    d.croots.push_back(r);
  }
  s->K0p = n_features <= 64 ? 64 : n_features <= 96 ? 96 : n_features <= 128 ? 128 : 256;
  build_round_tables(d, s->rt);
  return s;
}

// ============================================================================ C ABI
#define FELIX_API_BEGIN try {
#define FELIX_API_END                                                   \
  }                                                                     \
  catch (const felix::Error& e) { felix::set_error(e.msg); return e.code; } \
  catch (const std::bad_alloc&) { felix::set_error("host allocation failed"); return FELIX_E_OOM; } \
  catch (const std::exception& e) { felix::set_error(e.what()); return FELIX_E_CUDA; } \
  return FELIX_OK;

extern "C" {

const char* felix_last_error(void) { return g_last_error.c_str(); }

felix_status felix_merge_topk(const int64_t* key, const double* score, const int32_t* sched, int64_t n_rows,
                              int32_t n_vars, int32_t k, int64_t* key_out, double* score_out, int32_t* sched_out,
                              int32_t* n_out) {
  FELIX_API_BEGIN
  if (n_vars < 1 || k < 0 || n_rows < 0 || !n_out) FELIX_THROW(FELIX_E_INVALID_ARG, "felix_merge_topk: bad sizes");
  if (n_rows > 0 && (!key || !score || !sched)) FELIX_THROW(FELIX_E_INVALID_ARG, "felix_merge_topk: NULL input");
  if (k > 0 && (!key_out || !score_out || !sched_out)) FELIX_THROW(FELIX_E_INVALID_ARG, "felix_merge_topk: NULL output");
  std::vector<int64_t> rows;
  for (int64_t r = 0; r < n_rows; ++r) if (key[r] >= 0) rows.push_back(r);
  // (score desc, key asc); NaN scores after every number
  std::sort(rows.begin(), rows.end(), [&](int64_t a, int64_t b) {
    const bool na = std::isnan(score[a]), nb = std::isnan(score[b]);
    if (na != nb) return nb;
    if (!na && score[a] != score[b]) return score[a] > score[b];
    return key[a] < key[b];
  });
  std::set<std::vector<int32_t>> seen;
  int32_t m = 0;
  for (int64_t r : rows) {
    if (m >= k) break;
    std::vector<int32_t> sv(sched + r * n_vars, sched + (r + 1) * n_vars);
    if (!seen.insert(sv).second) continue;
    key_out[m] = key[r];
    score_out[m] = score[r];
    std::copy(sv.begin(), sv.end(), sched_out + static_cast<int64_t>(m) * n_vars);
    ++m;
  }
  *n_out = m;
  FELIX_API_END
}
int32_t felix_abi_version(void) { return FELIX_ABI_VERSION; }

felix_status felix_space_create(int device, const felix_var* vars, int32_t n_vars, const felix_split* splits,
                                int32_t n_splits, const felix_node* nodes, int32_t n_nodes, const int32_t* feature_roots,
                                int32_t n_features, const int32_t* constraint_roots, int32_t n_constraints,
                                felix_space** out) {
  FELIX_API_BEGIN
  if (!out) FELIX_THROW(FELIX_E_INVALID_ARG, "out is NULL");
  *out = nullptr;
  auto s = parse_space(vars, n_vars, splits, n_splits, nodes, n_nodes, feature_roots, n_features, constraint_roots,
                       n_constraints);
  s->device = device;
  check_device(device);
  DeviceGuard dg(device);
  const auto& t = s->rt;
  upload(s->d_comp_nvars, t.comp_nvars); upload(s->d_comp_var0, t.comp_var0); upload(s->d_comp_vars, t.comp_vars);
  upload(s->d_comp_eoff, t.comp_eoff); upload(s->d_comp_tcount, t.comp_tcount);
  upload(s->d_tuples, t.tuples); upload(s->d_lnf, t.lnf);
  std::vector<int32_t> iv(t.int_vars.begin(), t.int_vars.end());
  std::vector<int64_t> icnt;
  for (size_t q = 0; q < t.int_vars.size(); ++q) icnt.push_back(t.int_hi[q] - t.int_lo[q]);
  upload(s->d_int_vars, iv); upload(s->d_int_lo, t.int_lo); upload(s->d_int_cnt, icnt);
  upload(s->d_int_toff, t.int_toff); upload(s->d_int_thr, t.int_thr);
  upload(s->d_comp_ns, t.comp_ns); upload(s->d_comp_s0, t.comp_s0); upload(s->d_comp_sext, t.comp_sext);
  upload(s->d_var_smask, t.var_smask); upload(s->d_var_doff, t.var_doff); upload(s->d_var_dcnt, t.var_dcnt);
  upload(s->d_dval, t.dval); upload(s->d_dln, t.dln); upload(s->d_bnb_sel, t.bnb_comps);
  std::vector<int32_t> all_sel(t.comp_nvars.size());
  std::iota(all_sel.begin(), all_sel.end(), 0);
  upload(s->d_all_sel, all_sel);
  get_module(s.get(), 1);
  *out = s.release();
  FELIX_API_END
}


felix_status felix_codegen(const felix_var* vars, int32_t n_vars, const felix_split* splits, int32_t n_splits,
                           const felix_node* nodes, int32_t n_nodes, const int32_t* feature_roots, int32_t n_features,
                           const int32_t* constraint_roots, int32_t n_constraints, int32_t n_statements,
                           int32_t compile, char* src, int64_t src_cap, int64_t* src_len) {
  FELIX_API_BEGIN
  auto s = parse_space(vars, n_vars, splits, n_splits, nodes, n_nodes, feature_roots, n_features, constraint_roots,
                       n_constraints);
  if (n_statements < 1 || n_features % n_statements != 0 || n_features / n_statements > 128)
    FELIX_THROW(FELIX_E_INVALID_ARG, "n_statements must divide n_features into vectors of <= 128");
  s->desc.n_statements = n_statements;
  const int K0 = n_features / n_statements;
  s->K0p = K0 <= 64 ? 64 : K0 <= 96 ? 96 : 128;
  CodegenInfo info;
  // felix_tune("codegen_cone_width" / "codegen_replicas") select the variant to inspect (default P = 4, R = 2)
  const int cp = g_tune.codegen_P.load(), cr = g_tune.codegen_R.load();
  const std::string code = generate_dag_module(s->desc, s->K0p, cp > 0 ? cp : 4, cr > 0 ? cr : 2, g_tune.trace.load() != 0, 1, &info);
  if (src_len) *src_len = static_cast<int64_t>(code.size());
  if (src && src_cap > 0) {
    const size_t nb = std::min<size_t>(code.size() + 1, static_cast<size_t>(src_cap));
    std::memcpy(src, code.c_str(), nb);
  }
  if (compile) (void)compile_module_parts(code);
  FELIX_API_END
}

void felix_space_destroy(felix_space* s) {
  if (!s) return;
  int prev = -1;
  cudaGetDevice(&prev);
  cudaSetDevice(s->device);
  delete s;
  if (prev >= 0) cudaSetDevice(prev);
}

felix_status felix_space_set_statements(felix_space* s, int32_t n_statements) {
  FELIX_API_BEGIN
  if (!s) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL space");
  const int K = static_cast<int>(s->desc.froots.size());
  if (n_statements < 1 || K % n_statements != 0)
    FELIX_THROW(FELIX_E_INVALID_ARG, "n_statements must divide n_features");
  const int K0 = K / n_statements;
  if (K0 > 128) FELIX_THROW(FELIX_E_UNSUPPORTED, "per-statement feature width > 128");
  DeviceGuard dg(s->device);
  CUDA_OK(cudaDeviceSynchronize());
  s->desc.n_statements = n_statements;
  s->K0p = K0 <= 64 ? 64 : K0 <= 96 ? 96 : 128;
  for (auto& kv : s->modules)
    for (cudaLibrary_t l : kv.second.libs) if (l) cudaLibraryUnload(l);
  s->modules.clear();
  s->search_chunks.reset();
  s->eval_chunks.reset();
  s->group_cache.reset();
  s->uid = next_uid();   // group caches on other spaces that list this one become stale
  FELIX_API_END
}

felix_status felix_space_info(const felix_space* s, felix_space_info_t* out) {
  FELIX_API_BEGIN
  if (!s || !out) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL argument");
  out->n_vars = s->desc.n_vars;
  out->n_nodes = static_cast<int32_t>(s->desc.nodes.size());
  out->n_features = static_cast<int32_t>(s->desc.froots.size());
  out->n_constraints_user = static_cast<int32_t>(s->desc.croots.size());
  out->n_roots_total = s->desc.n_roots_total();
  out->n_components = static_cast<int32_t>(s->rt.comp_nvars.size());
  out->n_tuples_total = s->rt.n_tuples_total;
  out->nvrtc_ms = s->nvrtc_ms;
  out->regs_fwd = s->regs_fwd;
  out->regs_rev = s->regs_rev;
  out->dag_flops_fwd = s->flops_fwd;
  out->dag_flops_rev = s->flops_rev;
  FELIX_API_END
}

static void split_half(const std::vector<float>& x, std::vector<__half>& hi, std::vector<__half>& lo) {
  hi.resize(x.size());
  lo.resize(x.size());
  for (size_t i = 0; i < x.size(); ++i) {
    hi[i] = __float2half_rn(x[i]);
    lo[i] = __float2half_rn(x[i] - __half2float(hi[i]));
  }
}

felix_status felix_costmodel_load(int device, int32_t n_layers, const int32_t* dims, const float* const* W,
                                  const float* const* b, felix_costmodel** out) {
  FELIX_API_BEGIN
  if (!out || !dims || !W || !b) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL argument");
  *out = nullptr;
  if (n_layers < 2 || n_layers > 16) FELIX_THROW(FELIX_E_UNSUPPORTED, "n_layers must be in [2, 16]");
  if (dims[n_layers] != 1) FELIX_THROW(FELIX_E_SHAPE, "the last layer must have one output (predicted performance)");
  if (dims[0] < 1 || dims[0] > 256) FELIX_THROW(FELIX_E_UNSUPPORTED, "dims[0] must be in [1, 256]");
  for (int l = 1; l < n_layers; ++l)
    if (dims[l] <= 0 || dims[l] % 64 != 0 || dims[l] > CHAIN_MAX_N) FELIX_THROW(FELIX_E_UNSUPPORTED, "hidden dims must be multiples of 64 in [64, 1024]");
  for (int l = 0; l < n_layers; ++l) if (!W[l] || !b[l]) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL weight");
  check_device(device);
  DeviceGuard dg(device);
  auto m = std::make_unique<felix_costmodel>();
  m->uid = next_uid();
  m->device = device;
  m->n_layers = n_layers;
  m->dims.assign(dims, dims + n_layers + 1);
  m->K0p = dims[0] <= 64 ? 64 : dims[0] <= 96 ? 96 : dims[0] <= 128 ? 128 : 256;
  for (int l = 0; l < n_layers - 1; ++l) {
    const int N = dims[l + 1], K = dims[l];
    const int Kp = (l == 0) ? m->K0p : K;
    std::vector<float> w(static_cast<size_t>(N) * Kp, 0.f), wt(static_cast<size_t>(Kp) * N, 0.f);
    for (int r = 0; r < N; ++r)
      for (int c = 0; c < K; ++c) {
        const float v = W[l][static_cast<size_t>(r) * K + c];
        w[static_cast<size_t>(r) * Kp + c] = v;
        wt[static_cast<size_t>(c) * N + r] = v;
      }
    std::vector<__half> hi, lo, thi, tlo;
    split_half(w, hi, lo);
    split_half(wt, thi, tlo);
    for (auto* vec : {&m->W_hi, &m->W_lo, &m->WT_hi, &m->WT_lo, &m->bias}) vec->push_back(std::make_unique<DevBuf>());
    upload(*m->W_hi.back(), hi); upload(*m->W_lo.back(), lo);
    upload(*m->WT_hi.back(), thi); upload(*m->WT_lo.back(), tlo);
    upload(*m->bias.back(), std::vector<float>(b[l], b[l] + N));
  }
  const int Dh = dims[n_layers - 1];
  upload(m->head_w, std::vector<float>(W[n_layers - 1], W[n_layers - 1] + Dh));
  if (n_layers >= 2) {
    const int l = n_layers - 2, N = dims[l + 1], K = dims[l];
    const int Kp = (l == 0) ? m->K0p : K;
    std::vector<float> wt(static_cast<size_t>(Kp) * N, 0.f);
    for (int r = 0; r < N; ++r)
      for (int c = 0; c < K; ++c)
        wt[static_cast<size_t>(c) * N + r] = -W[n_layers - 1][r] * W[l][static_cast<size_t>(r) * K + c];
    std::vector<__half> thi, tlo;
    split_half(wt, thi, tlo);
    upload(m->WTs_hi, thi);
    upload(m->WTs_lo, tlo);
  }
  m->head_b = b[n_layers - 1][0];
  for (int l = 0; l < n_layers; ++l) {
    const int N = dims[l + 1], K = dims[l];
    std::vector<double> w64(W[l], W[l] + static_cast<size_t>(N) * K), b64(b[l], b[l] + N);
    m->W64.push_back(std::make_unique<DevBuf>());
    m->b64.push_back(std::make_unique<DevBuf>());
    upload(*m->W64.back(), w64);
    upload(*m->b64.back(), b64);
  }
  *out = m.release();
  FELIX_API_END
}

void felix_costmodel_destroy(felix_costmodel* m) { delete m; }

static void check_pair(felix_space* s, felix_costmodel* m) {
  if (!s || !m) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL handle");
  if (s->desc.k0() != m->dims[0])
    FELIX_THROW(FELIX_E_SHAPE, "space per-statement n_features != cost model dims[0]");
  if (s->device != m->device) FELIX_THROW(FELIX_E_INVALID_ARG, "space and cost model on different devices");
}

static void do_round(felix_space* s, const float* y, int64_t n, int32_t* sched, cudaStream_t st);

felix_status felix_search(felix_space* s, felix_costmodel* m, const felix_search_params* p, float* y,
                          float* final_loss, void* stream) {
  FELIX_API_BEGIN
  check_pair(s, m);
  if (!p) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL params");
  if (p->n_seeds == 0) return FELIX_OK;
  if (!y) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL y");
  if (p->n_seeds < 0 || p->n_seeds > (int64_t(1) << 30)) FELIX_THROW(FELIX_E_INVALID_ARG, "n_seeds out of range");
  if (p->n_steps < 0) FELIX_THROW(FELIX_E_INVALID_ARG, "n_steps < 0");
  if (p->n_seeds == 0) return FELIX_OK;
  DeviceGuard dg(s->device);
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const int64_t n = p->n_seeds;
  Chunks& ch = get_chunks(s, s->search_chunks, m, n, choose_chunks(n));
  const int nck = static_cast<int>(ch.plans.size());
  const bool sc = use_sc() && !p->history;
  const int P0 = choose_P(ch.cnt[0]);
  const int dpp = ch.plans[0]->dphi_parts;
  const felix_space::Module& mod = sc ? get_module(s, choose_P_sc(P0), choose_R_sc(), dpp) : get_module(s, P0, choose_R(ch.cnt[0], P0), dpp);
  const int scw = choose_scw(ch.cnt[0], mod.P);
  if (!p->init_from_y) {
    unsigned long long seed = p->rng_seed;
    long long ib = p->index_base;
    int ni = static_cast<int>(n);
    void* args[] = {&seed, &ni, &ib, &y};
    prof_mark(s, 3, st, true);
    launch_warp_per_item(mod.f_init, n, args, st);
    prof_mark(s, 3, st, false);
    s->prof_launches[3] += 1;
  }
  for (auto& pl : ch.plans) {
    CUDA_OK(cudaMemsetAsync(pl->m.p, 0, pl->m.bytes, st));
    CUDA_OK(cudaMemsetAsync(pl->v.p, 0, pl->v.bytes, st));
    CUDA_OK(cudaMemsetAsync(pl->step_ctr.p, 0, 4, st));
    // the grid-barrier counter's target arithmetic is not wrap-safe (2^32 is not a multiple of the grid):
    // restart it every search (stream-ordered, no chain kernel in flight on this workspace)
    CUDA_OK(cudaMemsetAsync(pl->grid_bar.p, 0, pl->grid_bar.bytes, st));
    // dataflow flags count up with step_ctr (reset together; 8 * steps stays far below 2^32)
    CUDA_OK(cudaMemsetAsync(pl->chain_flags.p, 0, pl->chain_flags.bytes, st));
    if (sc) {
      const int64_t cnt = pl->n / s->desc.n_statements;
      ensure(pl->sc_part, static_cast<size_t>(mod.P) * s->desc.n_vars * cnt * 4);
      ensure(pl->sc_pen, static_cast<size_t>(mod.P) * cnt * 8);
      set_int_kernel<<<1, 1, 0, st>>>(pl->step_ctr.as<int>(), 1);   // the reverse kernel counts from 1
      CUDA_OK(cudaGetLastError());
      s->prof_launches[3] += 1;
    }
  }
  // varValuesHistory: a fresh pool for this search (worst case: every seed at every step is new)
  const int M = s->desc.n_vars;
  s->h_valid = p->history != 0;
  if (s->h_valid) {
    const int64_t cap = n * std::max(1, p->n_steps);
    if (cap > INT32_MAX - 1) FELIX_THROW(FELIX_E_UNSUPPORTED, "history: n_seeds x n_steps exceeds 2^31 schedules");
    uint64_t slots = 1024;
    while (slots < static_cast<uint64_t>(cap) * 2) slots <<= 1;
    ensure(s->h_sched, static_cast<size_t>(n) * M * 4);
    ensure(s->h_last, static_cast<size_t>(n) * M * 4);
    ensure(s->h_slot_h, slots * 8);
    ensure(s->h_slot_i, slots * 4);
    ensure(s->h_pool_sched, static_cast<size_t>(cap) * M * 4);
    ensure(s->h_pool_key, static_cast<size_t>(cap) * 8);
    ensure(s->h_cnt, 8);
    CUDA_OK(cudaMemsetAsync(s->h_slot_h.p, 0, slots * 8, st));
    CUDA_OK(cudaMemsetAsync(s->h_slot_i.p, 0xFF, slots * 4, st));
    CUDA_OK(cudaMemsetAsync(s->h_cnt.p, 0, 8, st));
    s->h_n = n;
    s->h_cap = cap;
    s->h_mask = slots - 1;
    s->h_index_base = p->index_base;
  }
  // round sigma_x_i (before this step's fwd kernel bumps step_ctr) and insert new schedules
  auto history_step = [&](cudaStream_t cs) {
    do_round(s, y, n, s->h_sched.as<int32_t>(), cs);
    hist_insert_kernel<<<static_cast<unsigned>((n + 255) / 256), 256, 0, cs>>>(
        s->h_sched.as<int32_t>(), static_cast<int>(n), M, ch.plans[0]->step_ctr.as<int>(), s->h_last.as<int32_t>(),
        s->h_slot_h.as<unsigned long long>(), s->h_slot_i.as<int>(), s->h_mask, s->h_pool_sched.as<int32_t>(),
        s->h_pool_key.as<long long>(), s->h_cnt.as<int>(), static_cast<int>(s->h_cap), s->h_cnt.as<int>() + 1);
    CUDA_OK(cudaGetLastError());
  };
  const float hb = m->head_b, lam0 = p->lambda, lr0 = p->lr, b10 = p->beta1, b20 = p->beta2, eps0 = p->eps;
  // one Adam step of chunk k (fwd DAG -> GEMMs -> reverse DAG + Adam), PDL-chained on stream cs
  auto chunk_step = [&](int k, cudaStream_t cs) {
    Plan& pl = *ch.plans[k];
    const int64_t o = ch.off[k], cnt = ch.cnt[k];
    float* yk = y + o;
    int* ctr = pl.step_ctr.as<int>();
    int ni = static_cast<int>(cnt), ldy = static_cast<int>(n);
    void* dphi = pl.dphi.p;
    void* cpart = pl.c_part.p;
    int ld = static_cast<int>(pl.n_pad);
    int nht = pl.n_head_tiles;
    float hbv = hb, lam = lam0, lr = lr0, b1 = b10, b2 = b20, eps = eps0;
    void* mv = pl.m.p;
    void* vv = pl.v.p;
    if (sc) {
      // Adam step t-1 (in place) + features at y -> MLP -> split-cone reverse (partial adjoints)
      void* phh = pl.phi_hi.p;
      void* phl = pl.phi_lo.p;
      void* part = pl.sc_part.p;
      void* pen = pl.sc_pen.p;
      void* fa[] = {&yk, &ni, &ldy, &phh, &phl, &ctr, &mv, &vv, &part, &pen, &cpart, &nht, &ld, &hbv, &lam, &lr, &b1, &b2, &eps};
      prof_mark(s, 0, cs, true);
      launch_grouped(mod.f_fwd_adam, mod.P, mod.R, cnt, 0, fa, cs, pdl_mask() & 1);   // default: no PDL edge from the previous step's reverse (measured slower)
      prof_mark(s, 0, cs, false);
      s->prof_launches[0] += 1;
      run_mlp(s, pl, cs);
      void* ra[] = {&yk, &ni, &ldy, &dphi, &ld, &lam, &part, &pen, &ctr};
      prof_mark(s, 2, cs, true);
      launch_sc(mod.f_rev_sc, mod.P, scw, cnt, ra, cs, (pdl_mask() & 4) != 0);
      prof_mark(s, 2, cs, false);
      s->prof_launches[2] += 1;
      return;
    }
    run_forward_mlp(s, pl, mod, yk, cnt, n, cs, ctr);
    float* lo = final_loss ? final_loss + o : nullptr;   // every step writes its loss; the last one stays
    void* args[] = {&yk, &ni, &ldy, &dphi, &ld, &cpart, &nht, &ld, &hbv, &lam, &mv, &vv, &ctr, &lr, &b1, &b2, &eps, &lo};
    prof_mark(s, 2, cs, true);
    launch_grouped(mod.f_rev_adam, mod.P, mod.R, cnt, mod.rev_smem, args, cs, true);
    prof_mark(s, 2, cs, false);
    s->prof_launches[2] += 1;
  };
  if (s->profiling) {
    for (int t = 1; t <= p->n_steps; ++t) {          // direct launches with per-class events
      if (s->h_valid) {
        prof_mark(s, 3, st, true);
        history_step(st);
        prof_mark(s, 3, st, false);
      }
      for (int k = 0; k < nck; ++k) chunk_step(k, st);
    }
  } else if (p->n_steps > 0 && nck > 1 && !s->h_valid) {
    // The chunks are independent candidates: each gets its own one-step graph on its own stream,
    // launched n_steps times with no per-step join, so one chunk's MLP overlaps another's DAG kernels
    // (a per-step fork/join would re-synchronise them every step).  Joined once at the end.
    auto ptr = [](const void* q) { return static_cast<double>(reinterpret_cast<uintptr_t>(q)); };
    const std::vector<double> key = {static_cast<double>(mod.P), ptr(y), ptr(final_loss), lam0, lr0, b10, b20, eps0,
                                     static_cast<double>(sc), static_cast<double>(scw), static_cast<double>(mod.R),
                                     ptr(ch.plans[0]->sc_part.p), ptr(ch.plans[0]->sc_pen.p)};
    while (static_cast<int>(ch.streams.size()) < nck) {
      cudaStream_t b;
      CUDA_OK(cudaStreamCreateWithFlags(&b, cudaStreamNonBlocking));
      ch.streams.push_back(b);
    }
    if (!ch.ev_fork) CUDA_OK(cudaEventCreateWithFlags(&ch.ev_fork, cudaEventDisableTiming));
    while (static_cast<int>(ch.ev_join.size()) < nck) {
      cudaEvent_t e;
      CUDA_OK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
      ch.ev_join.push_back(e);
    }
    if (static_cast<int>(ch.chunk_graphs.size()) != nck || ch.chunk_key != key) {
      for (auto g : ch.chunk_graphs) if (g) cudaGraphExecDestroy(g);
      ch.chunk_graphs.assign(nck, nullptr);
      int64_t saved[4];
      std::copy(s->prof_launches, s->prof_launches + 4, saved);
      for (int k = 0; k < nck; ++k) {
        cudaGraph_t graph = nullptr;
        cudaStream_t cs = ch.streams[k];
        CUDA_OK(cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal));
        try {
          chunk_step(k, cs);
        } catch (...) {
          cudaStreamEndCapture(cs, &graph);
          if (graph) cudaGraphDestroy(graph);
          throw;
        }
        CUDA_OK(cudaStreamEndCapture(cs, &graph));
        cudaError_t ie = cudaGraphInstantiate(&ch.chunk_graphs[k], graph, 0);
        cudaGraphDestroy(graph);
        CUDA_OK(ie);
      }
      std::copy(saved, saved + 4, s->prof_launches);
      ch.chunk_key = key;
    }
    CUDA_OK(cudaEventRecord(ch.ev_fork, st));
    for (int k = 0; k < nck; ++k) CUDA_OK(cudaStreamWaitEvent(ch.streams[k], ch.ev_fork, 0));
    for (int t = 1; t <= p->n_steps; ++t)
      for (int k = 0; k < nck; ++k) CUDA_OK(cudaGraphLaunch(ch.chunk_graphs[k], ch.streams[k]));
    for (int k = 0; k < nck; ++k) {
      CUDA_OK(cudaEventRecord(ch.ev_join[k], ch.streams[k]));
      CUDA_OK(cudaStreamWaitEvent(st, ch.ev_join[k], 0));
    }
    s->prof_launches[0] += static_cast<int64_t>(p->n_steps) * nck;
    s->prof_launches[1] += static_cast<int64_t>(p->n_steps) * nck *
                           (ch.plans[0]->mode == MLP_LAYERS ? static_cast<int64_t>(ch.plans[0]->gemms.size()) : 1);
    s->prof_launches[2] += static_cast<int64_t>(p->n_steps) * nck;
  } else if (p->n_steps > 0) {
    auto ptr = [](const void* q) { return static_cast<double>(reinterpret_cast<uintptr_t>(q)); };
    const std::vector<double> key = {static_cast<double>(mod.P), ptr(y), ptr(final_loss), lam0, lr0, b10, b20, eps0,
                                     static_cast<double>(s->h_valid), ptr(s->h_sched.p), ptr(s->h_last.p),
                                     ptr(s->h_slot_h.p), ptr(s->h_pool_sched.p), ptr(s->h_pool_key.p),
                                     static_cast<double>(s->h_mask), static_cast<double>(s->h_cap),
                                     static_cast<double>(sc), static_cast<double>(scw), static_cast<double>(mod.R),
                                     ptr(ch.plans[0]->sc_part.p), ptr(ch.plans[0]->sc_pen.p)};
    // Several Adam steps per graph: inside one graph the programmatic (PDL) edges also link step t's
    // reverse kernel to step t+1's forward, and the graph launch cost is paid once per kGraphSteps steps
    // (between graph launches the next step waits for the whole previous graph).
    auto build = [&](int steps) {
      while (static_cast<int>(ch.streams.size()) < nck) {
        cudaStream_t b;
        CUDA_OK(cudaStreamCreateWithFlags(&b, cudaStreamNonBlocking));
        ch.streams.push_back(b);
      }
      cudaGraph_t graph = nullptr;
      cudaGraphExec_t exec = nullptr;
      cudaEvent_t fork, join[16];
      CUDA_OK(cudaEventCreateWithFlags(&fork, cudaEventDisableTiming));
      for (int k = 0; k < nck; ++k) CUDA_OK(cudaEventCreateWithFlags(&join[k], cudaEventDisableTiming));
      cudaStream_t cap = ch.streams[0];
      CUDA_OK(cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal));
      int64_t saved[4];
      std::copy(s->prof_launches, s->prof_launches + 4, saved);
      try {
        for (int i = 0; i < steps; ++i) {
          if (s->h_valid) history_step(cap);
          if (nck > 1) {
            CUDA_OK(cudaEventRecord(fork, cap));
            for (int k = 1; k < nck; ++k) CUDA_OK(cudaStreamWaitEvent(ch.streams[k], fork, 0));
          }
          for (int k = 0; k < nck; ++k) chunk_step(k, ch.streams[k]);
          for (int k = 1; k < nck; ++k) {
            CUDA_OK(cudaEventRecord(join[k], ch.streams[k]));
            CUDA_OK(cudaStreamWaitEvent(cap, join[k], 0));
          }
        }
        std::copy(saved, saved + 4, s->prof_launches);
      } catch (...) {
        cudaStreamEndCapture(cap, &graph);
        if (graph) cudaGraphDestroy(graph);
        cudaEventDestroy(fork);
        for (int k = 0; k < nck; ++k) cudaEventDestroy(join[k]);
        throw;
      }
      CUDA_OK(cudaStreamEndCapture(cap, &graph));
      cudaError_t ie = cudaGraphInstantiate(&exec, graph, 0);
      cudaGraphDestroy(graph);
      cudaEventDestroy(fork);
      for (int k = 0; k < nck; ++k) cudaEventDestroy(join[k]);
      CUDA_OK(ie);
      return exec;
    };
    const int gs_t = g_tune.graph_steps.load();
    const int gs = static_cast<int>(std::min<int64_t>(gs_t >= 1 ? gs_t : kGraphSteps, p->n_steps));
    const int tail = static_cast<int>(p->n_steps % gs);
    std::vector<double> key_s = key;
    key_s.push_back(static_cast<double>(gs));
    key_s.push_back(static_cast<double>(pdl_mask()));
    if (!ch.graph || ch.graph_key != key_s) {
      if (ch.graph) { cudaGraphExecDestroy(ch.graph); ch.graph = nullptr; }
      if (ch.graph_tail) { cudaGraphExecDestroy(ch.graph_tail); ch.graph_tail = nullptr; }
      ch.graph_tail_steps = 0;
      ch.graph = build(gs);
      ch.graph_key = key_s;
    }
    if (tail > 0 && (ch.graph_tail_steps != tail || !ch.graph_tail)) {
      if (ch.graph_tail) { cudaGraphExecDestroy(ch.graph_tail); ch.graph_tail = nullptr; }
      ch.graph_tail = build(tail);
      ch.graph_tail_steps = tail;
    }
    for (int64_t t = 0; t + gs <= p->n_steps; t += gs) {
      if (t % 100000 < gs && t > 0)   // keep the grid-barrier counter far from 2^32 on very long searches
        for (auto& pl : ch.plans) CUDA_OK(cudaMemsetAsync(pl->grid_bar.p, 0, pl->grid_bar.bytes, st));
      CUDA_OK(cudaGraphLaunch(ch.graph, st));
    }
    if (tail > 0) CUDA_OK(cudaGraphLaunch(ch.graph_tail, st));
    s->prof_launches[0] += static_cast<int64_t>(p->n_steps) * nck;
    s->prof_launches[1] += static_cast<int64_t>(p->n_steps) * nck *
                           (ch.plans[0]->mode == MLP_LAYERS ? static_cast<int64_t>(ch.plans[0]->gemms.size()) : 1);
    s->prof_launches[2] += static_cast<int64_t>(p->n_steps) * nck;
  }
  if (sc && p->n_steps > 0) {
    // the last Adam step (the forward kernel of step t applies step t-1) and the final loss
    for (int k = 0; k < nck; ++k) {
      Plan& pl = *ch.plans[k];
      const int64_t o = ch.off[k], cnt = ch.cnt[k];
      float* yk = y + o;
      int ni = static_cast<int>(cnt), ldy = static_cast<int>(n), ld = static_cast<int>(pl.n_pad), nht = pl.n_head_tiles;
      void* mv = pl.m.p;
      void* vv = pl.v.p;
      void* part = pl.sc_part.p;
      void* pen = pl.sc_pen.p;
      void* cpart = pl.c_part.p;
      void* ctr = pl.step_ctr.p;
      float* lo = final_loss ? final_loss + o : nullptr;
      float hbv = hb, lam = lam0, lr = lr0, b1 = b10, b2 = b20, eps = eps0;
      void* og = nullptr;
      void* aa[] = {&yk, &ni, &ldy, &mv, &vv, &part, &pen, &cpart, &nht, &ld, &hbv, &lam, &lr, &b1, &b2, &eps, &ctr, &lo, &og};
      prof_mark(s, 2, st, true);
      launch_flat(mod.f_adam_sc, cnt, aa, st);
      prof_mark(s, 2, st, false);
      s->prof_launches[2] += 1;
    }
  }
  FELIX_API_END
}

felix_status felix_search_group(felix_space* const* spaces, int32_t n_spaces, felix_costmodel* m,
                                const felix_search_params* params, float* const* y, float* const* final_loss, void* stream) {
  FELIX_API_BEGIN
  if (!spaces || !params || !y || n_spaces <= 0 || n_spaces > 256) FELIX_THROW(FELIX_E_INVALID_ARG, "bad group arguments");
  const int G = n_spaces;
  int64_t rows = 0;
  for (int i = 0; i < G; ++i) {
    check_pair(spaces[i], m);
    const felix_search_params& p = params[i];
    if (p.n_steps != params[0].n_steps) FELIX_THROW(FELIX_E_INVALID_ARG, "group members need equal n_steps");
    if (p.n_steps < 0) FELIX_THROW(FELIX_E_INVALID_ARG, "n_steps < 0");
    if (p.history) FELIX_THROW(FELIX_E_UNSUPPORTED, "history is not supported in group searches");
    if (p.n_seeds <= 0 || p.n_seeds > (int64_t(1) << 30)) FELIX_THROW(FELIX_E_INVALID_ARG, "n_seeds out of range");
    if (!y[i]) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL y");
    for (int j = 0; j < i; ++j) if (spaces[j] == spaces[i]) FELIX_THROW(FELIX_E_INVALID_ARG, "a space appears twice");
    rows += p.n_seeds * spaces[i]->desc.n_statements;
  }
  if (rows > (int64_t(1) << 30)) FELIX_THROW(FELIX_E_INVALID_ARG, "too many rows");
  felix_space* s0 = spaces[0];
  DeviceGuard dg(s0->device);
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const int T = params[0].n_steps;
  // ---- workspace (cached on spaces[0])
  std::unique_ptr<GroupCache>& slot = s0->group_cache;
  bool fresh = !slot || slot->cm_uid != m->uid || static_cast<int>(slot->space_uid.size()) != G;
  for (int i = 0; !fresh && i < G; ++i)
    fresh = slot->space_uid[i] != spaces[i]->uid || slot->space_ns[i] != spaces[i]->desc.n_statements ||
            slot->n[i] != params[i].n_seeds;
  if (fresh) {
    slot.reset();
    auto gc = std::make_unique<GroupCache>();
    gc->cm_uid = m->uid;
    int64_t off = 0;
    for (int i = 0; i < G; ++i) {
      gc->space_uid.push_back(spaces[i]->uid);
      gc->space_ns.push_back(spaces[i]->desc.n_statements);
      gc->n.push_back(params[i].n_seeds);
      gc->row_off.push_back(off);
      off += params[i].n_seeds * spaces[i]->desc.n_statements;
      for (auto* vec : {&gc->m, &gc->v}) {
        vec->push_back(std::make_unique<DevBuf>());
        vec->back()->alloc(static_cast<size_t>(spaces[i]->desc.n_vars) * params[i].n_seeds * 4);
      }
      gc->step_ctr.push_back(std::make_unique<DevBuf>());
      gc->step_ctr.back()->alloc(16);
      for (auto* vec : {&gc->sc_part, &gc->sc_pen}) vec->push_back(std::make_unique<DevBuf>());
    }
    gc->plan = build_plan_rows(s0->device, m, rows, 0, 0);
    gc->plan->chain.epoch = gc->step_ctr[0]->as<int>();   // every member's forward bumps its counter once per step
    for (int i = 0; i < G; ++i) {
      cudaStream_t b;
      CUDA_OK(cudaStreamCreateWithFlags(&b, cudaStreamNonBlocking));
      gc->streams.push_back(b);
    }
    slot = std::move(gc);
  }
  GroupCache& gc = *slot;
  Plan& pl = *gc.plan;
  // ---- per-search state: starting points, Adam state, counters, dataflow flags
  std::vector<const felix_space::Module*> mods(G);
  int64_t min_n = INT64_MAX;
  for (int i = 0; i < G; ++i) min_n = std::min<int64_t>(min_n, params[i].n_seeds);
  const bool sc = use_sc(true, min_n);
  std::vector<int> scws(G);
  for (int i = 0; i < G; ++i) {
    const int64_t n = params[i].n_seeds;
    mods[i] = sc ? &get_module(spaces[i], choose_P_sc(choose_P(n)), choose_R_sc(), pl.dphi_parts)
                 : &get_module(spaces[i], choose_P(n), choose_R(n, choose_P(n)), pl.dphi_parts);
    scws[i] = choose_scw(n, mods[i]->P);
    if (sc) {
      ensure(*gc.sc_part[i], static_cast<size_t>(mods[i]->P) * spaces[i]->desc.n_vars * n * 4);
      ensure(*gc.sc_pen[i], static_cast<size_t>(mods[i]->P) * n * 8);
    }
    if (!params[i].init_from_y) {
      unsigned long long seed = params[i].rng_seed;
      long long ib = params[i].index_base;
      int ni = static_cast<int>(n);
      float* yi = y[i];
      void* args[] = {&seed, &ni, &ib, &yi};
      launch_warp_per_item(mods[i]->f_init, n, args, st);
    }
    CUDA_OK(cudaMemsetAsync(gc.m[i]->p, 0, gc.m[i]->bytes, st));
    CUDA_OK(cudaMemsetAsync(gc.v[i]->p, 0, gc.v[i]->bytes, st));
    CUDA_OK(cudaMemsetAsync(gc.step_ctr[i]->p, 0, 4, st));
    if (sc) {
      set_int_kernel<<<1, 1, 0, st>>>(gc.step_ctr[i]->as<int>(), 1);   // the split-cone reverse counts from 1
      CUDA_OK(cudaGetLastError());
    }
  }
  CUDA_OK(cudaMemsetAsync(pl.grid_bar.p, 0, pl.grid_bar.bytes, st));
  CUDA_OK(cudaMemsetAsync(pl.chain_flags.p, 0, pl.chain_flags.bytes, st));
  if (T == 0) return FELIX_OK;
  // ---- one Adam step of every member: fork (DAG forwards write their phi rows at their row offsets),
  // join, one MLP pass over all rows, fork (reverse DAG + Adam per member on its dphi / head-partial
  // columns), join.  Captured once as a graph; with profiling on (spaces[0]) launched directly with
  // per-class events, the MLP as class 1.
  std::vector<cudaEvent_t> ev(2 * G + 2);
  for (auto& e : ev) CUDA_OK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  struct EvGuard { std::vector<cudaEvent_t>& v; ~EvGuard() { for (auto e : v) cudaEventDestroy(e); } } evg{ev};
  const int K0p = m->K0p;
  auto enqueue_step = [&](cudaStream_t main_st) {
    CUDA_OK(cudaEventRecord(ev[0], main_st));
    for (int i = 1; i < G; ++i) CUDA_OK(cudaStreamWaitEvent(gc.streams[i], ev[0], 0));
    for (int i = 0; i < G; ++i) {
      cudaStream_t si = i == 0 ? main_st : gc.streams[i];
      int ni = static_cast<int>(params[i].n_seeds), ldi = ni;
      const float* yi = y[i];
      void* phi_hi = pl.phi_hi.as<uint16_t>() + gc.row_off[i] * K0p;
      void* phi_lo = pl.phi_lo.as<uint16_t>() + gc.row_off[i] * K0p;
      int* ctr = gc.step_ctr[i]->as<int>();
      if (sc) {
        const felix_search_params& p = params[i];
        float* ya = y[i];
        void* mv = gc.m[i]->p;
        void* vv = gc.v[i]->p;
        void* part = gc.sc_part[i]->p;
        void* pen = gc.sc_pen[i]->p;
        void* cpart = pl.c_part.as<float>() + gc.row_off[i];
        int ld = static_cast<int>(pl.n_pad), nht = pl.n_head_tiles;
        float hbv = m->head_b, lam = p.lambda, lr = p.lr, b1 = p.beta1, b2 = p.beta2, eps = p.eps;
        void* fa[] = {&ya, &ni, &ldi, &phi_hi, &phi_lo, &ctr, &mv, &vv, &part, &pen, &cpart, &nht, &ld, &hbv, &lam, &lr, &b1, &b2, &eps};
        launch_grouped(mods[i]->f_fwd_adam, mods[i]->P, mods[i]->R, params[i].n_seeds, 0, fa, si, false);
        continue;
      }
      void* args[] = {&yi, &ni, &ldi, &phi_hi, &phi_lo, &ctr};
      launch_grouped(mods[i]->f_fwd, mods[i]->P, mods[i]->R, params[i].n_seeds, 0, args, si, false);
    }
    for (int i = 1; i < G; ++i) {
      CUDA_OK(cudaEventRecord(ev[1 + i], gc.streams[i]));
      CUDA_OK(cudaStreamWaitEvent(main_st, ev[1 + i], 0));
    }
    prof_mark(s0, 1, main_st, true);
    const MlpMode mode = static_cast<MlpMode>(pl.mode);
    if (mode == MLP_TILE) launch_tile(pl, main_st);
    else if (mode == MLP_CHAIN) launch_chain(pl, main_st);
    else for (const auto& g : pl.gemms) launch_gemm(g, main_st);
    prof_mark(s0, 1, main_st, false);
    CUDA_OK(cudaEventRecord(ev[G + 1], main_st));
    for (int i = 1; i < G; ++i) CUDA_OK(cudaStreamWaitEvent(gc.streams[i], ev[G + 1], 0));
    for (int i = 0; i < G; ++i) {
      cudaStream_t si = i == 0 ? main_st : gc.streams[i];
      const felix_search_params& p = params[i];
      float* yi = y[i];
      int ni = static_cast<int>(p.n_seeds), ldy = ni;
      void* dphi = pl.dphi.as<float>() + gc.row_off[i];
      void* cpart = pl.c_part.as<float>() + gc.row_off[i];
      int ld = static_cast<int>(pl.n_pad);
      int nht = pl.n_head_tiles;
      float hbv = m->head_b, lam = p.lambda, lr = p.lr, b1 = p.beta1, b2 = p.beta2, eps = p.eps;
      void* mv = gc.m[i]->p;
      void* vv = gc.v[i]->p;
      int* ctr = gc.step_ctr[i]->as<int>();
      float* lo = final_loss ? final_loss[i] : nullptr;
      if (sc) {
        void* part = gc.sc_part[i]->p;
        void* pen = gc.sc_pen[i]->p;
        void* ra[] = {&yi, &ni, &ldy, &dphi, &ld, &lam, &part, &pen, &ctr};
        launch_sc(mods[i]->f_rev_sc, mods[i]->P, scws[i], p.n_seeds, ra, si, false);
        continue;
      }
      void* args[] = {&yi, &ni, &ldy, &dphi, &ld, &cpart, &nht, &ld, &hbv, &lam, &mv, &vv, &ctr, &lr, &b1, &b2, &eps, &lo};
      launch_grouped(mods[i]->f_rev_adam, mods[i]->P, mods[i]->R, p.n_seeds, mods[i]->rev_smem, args, si, false);
    }
    for (int i = 1; i < G; ++i) {
      CUDA_OK(cudaEventRecord(ev[G + 1 + i], gc.streams[i]));
      CUDA_OK(cudaStreamWaitEvent(main_st, ev[G + 1 + i], 0));
    }
  };
  // the last Adam step of split-cone members (their forward kernel of step t applies step t-1)
  auto final_adam = [&]() {
    if (!sc) return;
    for (int i = 0; i < G; ++i) {
      const felix_search_params& p = params[i];
      float* ya = y[i];
      int ni = static_cast<int>(p.n_seeds), ldy = ni, ld = static_cast<int>(pl.n_pad), nht = pl.n_head_tiles;
      void* mv = gc.m[i]->p;
      void* vv = gc.v[i]->p;
      void* part = gc.sc_part[i]->p;
      void* pen = gc.sc_pen[i]->p;
      void* cpart = pl.c_part.as<float>() + gc.row_off[i];
      void* ctr = gc.step_ctr[i]->p;
      float* lo = final_loss ? final_loss[i] : nullptr;
      float hbv = m->head_b, lam = p.lambda, lr = p.lr, b1 = p.beta1, b2 = p.beta2, eps = p.eps;
      void* og = nullptr;
      void* aa[] = {&ya, &ni, &ldy, &mv, &vv, &part, &pen, &cpart, &nht, &ld, &hbv, &lam, &lr, &b1, &b2, &eps, &ctr, &lo, &og};
      launch_flat(mods[i]->f_adam_sc, p.n_seeds, aa, st);
    }
  };
  if (s0->profiling) {
    for (int t = 1; t <= T; ++t) {
      if (t % 100000 == 0) CUDA_OK(cudaMemsetAsync(pl.grid_bar.p, 0, pl.grid_bar.bytes, st));
      enqueue_step(st);
      s0->prof_launches[1] += 1;
    }
    final_adam();
    return FELIX_OK;
  }
  auto ptr = [](const void* q) { return static_cast<double>(reinterpret_cast<uintptr_t>(q)); };
  std::vector<double> key;
  for (int i = 0; i < G; ++i) {
    const felix_search_params& p = params[i];
    key.insert(key.end(), {static_cast<double>(mods[i]->P), static_cast<double>(mods[i]->R), ptr(y[i]),
                           ptr(final_loss ? final_loss[i] : nullptr), p.lambda, p.lr, p.beta1, p.beta2, p.eps,
                           static_cast<double>(sc), static_cast<double>(scws[i]), ptr(gc.sc_part[i]->p),
                           ptr(gc.sc_pen[i]->p)});
  }
  // several Adam steps per graph launch, as in felix_search
  auto build = [&](int steps) {
    cudaGraph_t graph = nullptr;
    cudaGraphExec_t exec = nullptr;
    cudaStream_t cap;
    CUDA_OK(cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking));
    struct StGuard { cudaStream_t s; ~StGuard() { cudaStreamDestroy(s); } } capg{cap};
    CUDA_OK(cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal));
    try {
      for (int i = 0; i < steps; ++i) enqueue_step(cap);
    } catch (...) {
      cudaStreamEndCapture(cap, &graph);
      if (graph) cudaGraphDestroy(graph);
      throw;
    }
    CUDA_OK(cudaStreamEndCapture(cap, &graph));
    cudaError_t ie = cudaGraphInstantiate(&exec, graph, 0);
    cudaGraphDestroy(graph);
    CUDA_OK(ie);
    return exec;
  };
  const int gs_t = g_tune.graph_steps.load();
  const int gs = std::max(1, std::min(gs_t >= 1 ? gs_t : kGraphSteps, T));
  const int tail = T > 0 ? T % gs : 0;
  key.push_back(static_cast<double>(gs));
  key.push_back(static_cast<double>(pdl_mask()));
  if (!gc.graph || gc.key != key) {
    if (gc.graph) { cudaGraphExecDestroy(gc.graph); gc.graph = nullptr; }
    if (gc.graph_tail) { cudaGraphExecDestroy(gc.graph_tail); gc.graph_tail = nullptr; }
    gc.graph_tail_steps = 0;
    gc.graph = build(gs);
    gc.key = key;
  }
  if (tail > 0 && (gc.graph_tail_steps != tail || !gc.graph_tail)) {
    if (gc.graph_tail) { cudaGraphExecDestroy(gc.graph_tail); gc.graph_tail = nullptr; }
    gc.graph_tail = build(tail);
    gc.graph_tail_steps = tail;
  }
  for (int t = 0; t + gs <= T; t += gs) {
    if (t % 100000 < gs && t > 0) CUDA_OK(cudaMemsetAsync(pl.grid_bar.p, 0, pl.grid_bar.bytes, st));
    CUDA_OK(cudaGraphLaunch(gc.graph, st));
  }
  if (tail > 0) CUDA_OK(cudaGraphLaunch(gc.graph_tail, st));
  final_adam();
  FELIX_API_END
}

// felix_eval / felix_eval_ex.  Default: one objective + gradient evaluation with the eval kernels
// (felix_fwd -> MLP -> felix_rev_eval).  search_path: the kernels and launch configuration of one
// felix_search Adam step (felix_fwd_adam at step 1, i.e. no update -> the MLP of the search plan ->
// felix_rev_sc partial adjoints -> felix_adam_sc summing them as the Adam prologue does), writing
// the loss and dL/dy instead of updating y.
static void eval_impl(felix_space* s, felix_costmodel* m, const float* y, int64_t n, float lambda, const felix_eval_out& o,
                      cudaStream_t st) {
  Plan& pl = *get_chunks(s, s->eval_chunks, m, n, 1).plans[0];
  CUDA_OK(cudaMemsetAsync(pl.grid_bar.p, 0, pl.grid_bar.bytes, st));
  CUDA_OK(cudaMemsetAsync(pl.chain_flags.p, 0, pl.chain_flags.bytes, st));
  CUDA_OK(cudaMemsetAsync(pl.step_ctr.p, 0, 4, st));     // the forward kernel makes it 1: the chain's epoch
  int ni = static_cast<int>(n);
  void* dphi = pl.dphi.p;
  void* cpart = pl.c_part.p;
  int ld = static_cast<int>(pl.n_pad);
  int nht = pl.n_head_tiles;
  float hb = m->head_b, lam = lambda;
  if (o.search_path) {
    const felix_space::Module& mod = get_module(s, choose_P_sc(choose_P(n)), choose_R_sc(), pl.dphi_parts);
    const int scw = choose_scw(n, mod.P);
    ensure(pl.sc_part, static_cast<size_t>(mod.P) * s->desc.n_vars * n * 4);
    ensure(pl.sc_pen, static_cast<size_t>(mod.P) * n * 8);
    CUDA_OK(cudaMemsetAsync(pl.m.p, 0, pl.m.bytes, st));
    CUDA_OK(cudaMemsetAsync(pl.v.p, 0, pl.v.bytes, st));
    set_int_kernel<<<1, 1, 0, st>>>(pl.step_ctr.as<int>(), 1);
    CUDA_OK(cudaGetLastError());
    float* yk = const_cast<float*>(y);   // step counter 1: felix_fwd_adam applies no update, y is not written
    int* ctr = pl.step_ctr.as<int>();
    void* phh = pl.phi_hi.p;
    void* phl = pl.phi_lo.p;
    void* part = pl.sc_part.p;
    void* pen = pl.sc_pen.p;
    void* mv = pl.m.p;
    void* vv = pl.v.p;
    float lr = 0.f, b1 = 0.9f, b2 = 0.999f, eps = 1e-8f;
    void* fa[] = {&yk, &ni, &ni, &phh, &phl, &ctr, &mv, &vv, &part, &pen, &cpart, &nht, &ld, &hb, &lam, &lr, &b1, &b2, &eps};
    launch_grouped(mod.f_fwd_adam, mod.P, mod.R, n, 0, fa, st, true);
    run_mlp(s, pl, st);
    void* ra[] = {&yk, &ni, &ni, &dphi, &ld, &lam, &part, &pen, &ctr};
    launch_sc(mod.f_rev_sc, mod.P, scw, n, ra, st, true);
    float* lo = o.loss;
    float* og = o.grad;
    void* aa[] = {&yk, &ni, &ni, &mv, &vv, &part, &pen, &cpart, &nht, &ld, &hb, &lam, &lr, &b1, &b2, &eps, &ctr, &lo, &og};
    launch_flat(mod.f_adam_sc, n, aa, st);
    return;
  }
  const felix_space::Module& mod = get_module(s, choose_P(n), choose_R(n, choose_P(n)), pl.dphi_parts);
  run_forward_mlp(s, pl, mod, y, n, n, st, pl.step_ctr.as<int>());
  float *phi = o.phi, *g = o.g, *cost = o.cost, *loss = o.loss, *grad = o.grad;
  double* F = o.F;
  void* args[] = {&y, &ni, &ni, &dphi, &ld, &cpart, &nht, &ld, &hb, &lam, &phi, &g, &cost, &loss, &grad, &F};
  launch_grouped(mod.f_rev_eval, mod.P, mod.R, n, mod.rev_smem, args, st, false);
}

felix_status felix_eval(felix_space* s, felix_costmodel* m, const float* y, int64_t n, float lambda, float* phi,
                        float* g, float* cost, float* loss, float* grad, void* stream) {
  felix_eval_out o{};
  o.phi = phi; o.g = g; o.cost = cost; o.loss = loss; o.grad = grad;
  return felix_eval_ex(s, m, y, n, lambda, &o, stream);
}

felix_status felix_eval_ex(felix_space* s, felix_costmodel* m, const float* y, int64_t n, float lambda,
                           const felix_eval_out* out, void* stream) {
  FELIX_API_BEGIN
  check_pair(s, m);
  if (!out) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL out");
  if (!y && n > 0) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL y");
  if (n < 0 || n > (int64_t(1) << 30)) FELIX_THROW(FELIX_E_INVALID_ARG, "n out of range");
  if (out->search_path && (out->phi || out->g || out->cost || out->F))
    FELIX_THROW(FELIX_E_INVALID_ARG, "search_path evaluates loss and grad only");
  if (n == 0) return FELIX_OK;
  DeviceGuard dg(s->device);
  eval_impl(s, m, y, n, lambda, *out, static_cast<cudaStream_t>(stream));
  FELIX_API_END
}

felix_status felix_init_sample(felix_space* s, int64_t n, uint64_t rng_seed, int64_t index_base, float* y, void* stream) {
  FELIX_API_BEGIN
  if (!s || (!y && n > 0)) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL argument");
  if (n < 0 || n > (int64_t(1) << 30)) FELIX_THROW(FELIX_E_INVALID_ARG, "n out of range");
  if (n == 0) return FELIX_OK;
  DeviceGuard dg(s->device);
  int ni = static_cast<int>(n);
  unsigned long long seed = rng_seed;
  long long ib = index_base;
  void* args[] = {&seed, &ni, &ib, &y};
  launch_warp_per_item(get_module(s, 1).f_init, n, args, static_cast<cudaStream_t>(stream));
  FELIX_API_END
}

static void do_round(felix_space* s, const float* y, int64_t n, int32_t* sched, cudaStream_t st) {
  const int M = s->desc.n_vars;
  const int nc = static_cast<int>(s->rt.comp_nvars.size());
  const int ni = static_cast<int>(n);
  const bool force_bnb = g_tune.round_bnb.load() != 0;
  if (nc > 0 && !force_bnb) {
    const long long warps = static_cast<long long>(n) * nc;
    const unsigned grid = static_cast<unsigned>((warps * 32 + 255) / 256);
    round_split_kernel<<<grid, 256, 0, st>>>(y, ni, M, nc, s->d_comp_nvars.as<int>(), s->d_comp_var0.as<int>(),
                                             s->d_comp_vars.as<int>(), s->d_comp_eoff.as<long long>(),
                                             s->d_comp_tcount.as<long long>(), s->d_tuples.as<int>(),
                                             s->d_lnf.as<double>(), sched);
    CUDA_OK(cudaGetLastError());
  }
  const int nb = force_bnb ? nc : static_cast<int>(s->rt.bnb_comps.size());
  if (nb > 0) {
    // warp per (candidate, component); the DP bound table of a single-split component ((nv + 1) x #divisors
    // doubles) sits in shared memory, up to 24 KB per warp (components above that use the weaker bound)
    int dp_cap = 0;
    for (int i = 0; i < nb; ++i) {
      const int c = force_bnb ? i : s->rt.bnb_comps[i];
      if (s->rt.comp_ns[c] != 1) continue;
      const int need = (s->rt.comp_nvars[c] + 1) * s->rt.var_dcnt[s->rt.comp_var0[c]] * 8;
      if (need <= 24576) dp_cap = std::max(dp_cap, need);
    }
    dp_cap = (dp_cap + 15) / 16 * 16;
    if (dp_cap * 4 > 48 * 1024) set_smem_attr(reinterpret_cast<const void*>(round_bnb_kernel), dp_cap * 4);
    const long long tot = static_cast<long long>(n) * nb * 32;
    round_bnb_kernel<<<static_cast<unsigned>((tot + 127) / 128), 128, dp_cap * 4, st>>>(
        y, ni, M, nb, (force_bnb ? s->d_all_sel : s->d_bnb_sel).as<int>(), s->d_comp_nvars.as<int>(),
        s->d_comp_var0.as<int>(), s->d_comp_vars.as<int>(), s->d_comp_ns.as<int>(), s->d_comp_s0.as<int>(),
        s->d_comp_sext.as<long long>(), s->d_var_smask.as<unsigned>(), s->d_var_doff.as<long long>(),
        s->d_var_dcnt.as<int>(), s->d_dval.as<long long>(), s->d_dln.as<double>(), sched, dp_cap);
    CUDA_OK(cudaGetLastError());
  }
  const int nint = static_cast<int>(s->rt.int_vars.size());
  if (nint > 0) {
    const long long tot = static_cast<long long>(n) * nint;
    round_int_kernel<<<static_cast<unsigned>((tot + 255) / 256), 256, 0, st>>>(
        y, ni, M, nint, s->d_int_vars.as<int>(), s->d_int_lo.as<long long>(), s->d_int_cnt.as<long long>(),
        s->d_int_toff.as<long long>(), s->d_int_thr.as<double>(), sched);
    CUDA_OK(cudaGetLastError());
  }
}

// Entries per block in the first top-k phase: every block selects its chunk's best k distinct schedules
// (k rounds of block argmax + dedup), the second phase merges the blocks' lists.  Enough blocks to run
// the rounds in parallel (C2: 8 blocks of 512 instead of one of 4096), few enough that the single-block
// merge stays short.
// one top-k selection phase: the shared-memory kernel when the block's entries fit (<= 96 KB), else the
// global-memory one (identical results)
static void launch_topk_select(long long nblk, long long n_entries, long long chunk, const int* cand_of,
                               const long long* okey, const double* score, const uint8_t* valid, const int32_t* sched,
                               int M, int k, uint8_t* alive, int* out_cand, int* out_cnt, cudaStream_t st) {
  const long long bytes = chunk * (8 + 8 + 4 + 4LL * M + 1);
  if (bytes <= 96 * 1024) {
    const int b = static_cast<int>((bytes + 15) / 16 * 16);
    if (b > 48 * 1024) set_smem_attr(reinterpret_cast<const void*>(topk_select_smem_kernel), 96 * 1024);
    topk_select_smem_kernel<<<static_cast<unsigned>(nblk), 1024, b, st>>>(n_entries, chunk, cand_of, okey, score, valid,
                                                                            sched, M, k, out_cand, out_cnt);
  } else {
    topk_select_kernel<<<static_cast<unsigned>(nblk), 1024, 0, st>>>(n_entries, chunk, cand_of, okey, score, valid,
                                                                       sched, M, k, alive, out_cand, out_cnt);
  }
  CUDA_OK(cudaGetLastError());
}

// Dedup + top-k of n entries in phases: each phase cuts its entries into blocks whose (score, key,
// candidate, schedule) fit shared memory and keeps each block's k best records; the records of one phase
// are the entries of the next, until one block remains.  Every phase is the same selection (score desc,
// key asc, dedup by schedule keeping the best), so the result equals a single pass over all entries.
static void run_topk(felix_space* s, int64_t n, const long long* okey, const int32_t* sched, int M, int k,
                     int* out_cand, int* out_cnt, cudaStream_t st);

static long long topk_chunk(long long n) {
  long long c = (n + 63) / 64;
  c = (c + 255) / 256 * 256;
  return std::max(512LL, std::min(4096LL, c));
}

static void run_topk(felix_space* s, int64_t n, const long long* okey, const int32_t* sched, int M, int k,
                     int* out_cand, int* out_cnt, cudaStream_t st) {
  const double* score = s->score.as<double>();
  const uint8_t* valid = s->valid.as<uint8_t>();
  long long chunk = 1;
  while (chunk * 2 * (8 + 8 + 4 + 4LL * M + 1) <= 96 * 1024) chunk *= 2;
  if (chunk < 2LL * k) {   // schedules too long for a shared-memory block of 2k entries: the global-memory kernel
    const long long ch = topk_chunk(n), nblk = (n + ch - 1) / ch;
    ensure(s->alive, static_cast<size_t>(std::max<long long>(n, nblk * k)));
    ensure(s->rec_cand, static_cast<size_t>(nblk) * k * 4);
    ensure(s->rec_cnt, static_cast<size_t>(nblk) * 4);
    launch_topk_select(nblk, n, ch, nullptr, okey, score, valid, sched, M, k, s->alive.as<uint8_t>(),
                       s->rec_cand.as<int>(), s->rec_cnt.as<int>(), st);
    launch_topk_select(1, nblk * k, nblk * k, s->rec_cand.as<int>(), okey, score, valid, sched, M, k,
                       s->alive.as<uint8_t>(), out_cand, out_cnt, st);
    return;
  }
  long long entries = n;
  const int* cand_of = nullptr;
  int phase = 0;
  while (true) {
    const long long nblk = (entries + chunk - 1) / chunk;
    int* oc;
    int* on;
    if (nblk == 1) {
      oc = out_cand;
      on = out_cnt;
    } else {
      felix::DevBuf& rc = (phase & 1) ? s->rec_cand2 : s->rec_cand;
      felix::DevBuf& rn = (phase & 1) ? s->rec_cnt2 : s->rec_cnt;
      ensure(rc, static_cast<size_t>(nblk) * k * 4);
      ensure(rn, static_cast<size_t>(nblk) * 4);
      oc = rc.as<int>();
      on = rn.as<int>();
    }
    launch_topk_select(nblk, entries, chunk, cand_of, okey, score, valid, sched, M, k, nullptr, oc, on, st);
    if (nblk == 1) return;
    cand_of = oc;
    entries = nblk * k;
    ++phase;
  }
}

static void do_hard(felix_space* s, const int32_t* sched, int64_t n, double* phi64, uint8_t* valid, cudaStream_t st) {
  int ni = static_cast<int>(n);
  void* args[] = {&sched, &ni, &phi64, &valid};
  launch_flat(get_module(s, 1).f_hard, n, args, st);
}


static void do_score(felix_space* s, felix_costmodel* m, const double* phi64, int64_t n, double* score, cudaStream_t st) {
  // TenSet segment sum over statements: score = sum_s MLP(phi_s), phi64 = [S * K0][n] statement-major
  const int L = m->n_layers;
  int maxw = 0;
  for (int l = 1; l < L; ++l) maxw = std::max(maxw, m->dims[l]);
  ensure(s->act64a, static_cast<size_t>(n) * maxw * 8);
  ensure(s->act64b, static_cast<size_t>(n) * maxw * 8);
  double* bufs[2] = {s->act64a.as<double>(), s->act64b.as<double>()};
  for (int st_i = 0; st_i < s->desc.n_statements; ++st_i) {
    const double* in = phi64 + static_cast<size_t>(st_i) * m->dims[0] * n;
    long long rs = 1, cs = n;    // phi64 is [K][n]
    for (int l = 0; l < L; ++l) {
      const int K = m->dims[l], N = m->dims[l + 1];
      const bool last = l == L - 1;
      double* out = last ? score : bufs[l & 1];
      if (N >= 32 && g_tune.score_dmma.load() != 0) {   // FP64 tensor cores, 128 x 64 tiles
        const long long big_tiles = ((N + SCD_TN - 1) / SCD_TN) * ((n + scd_tm<8>() - 1) / scd_tm<8>());
        if (big_tiles >= 2 * 148) {   // 256 x 64 tiles while they still give two per SM
          const dim3 grid(static_cast<unsigned>((N + SCD_TN - 1) / SCD_TN), static_cast<unsigned>((n + scd_tm<8>() - 1) / scd_tm<8>()));
          set_smem_attr(reinterpret_cast<const void*>(score_layer_dmma_kernel<8>), scd_smem<8>());
          score_layer_dmma_kernel<8><<<grid, 256, scd_smem<8>(), st>>>(
              in, rs, cs, static_cast<int>(n), K, m->W64[l]->as<double>(), m->b64[l]->as<double>(), out, N,
              last ? 0 : 1, last && st_i > 0 ? 1 : 0);
        } else {
          const dim3 grid(static_cast<unsigned>((N + SCD_TN - 1) / SCD_TN), static_cast<unsigned>((n + scd_tm<4>() - 1) / scd_tm<4>()));
          set_smem_attr(reinterpret_cast<const void*>(score_layer_dmma_kernel<4>), scd_smem<4>());
          score_layer_dmma_kernel<4><<<grid, 256, scd_smem<4>(), st>>>(
              in, rs, cs, static_cast<int>(n), K, m->W64[l]->as<double>(), m->b64[l]->as<double>(), out, N,
              last ? 0 : 1, last && st_i > 0 ? 1 : 0);
        }
      } else if (N >= 32) {   // register-blocked 128 x 64 tiles on the CUDA cores
        const dim3 grid(static_cast<unsigned>((N + SC2_TN - 1) / SC2_TN), static_cast<unsigned>((n + SC2_TM - 1) / SC2_TM));
        score_layer_v2_kernel<<<grid, 256, 0, st>>>(
            in, rs, cs, static_cast<int>(n), K, m->W64[l]->as<double>(), m->b64[l]->as<double>(), out, N,
            last ? 0 : 1, last && st_i > 0 ? 1 : 0);
      } else if (N == 1 && last && rs == K && cs == 1) {
        score_head_kernel<<<static_cast<unsigned>((n + 31) / 32), 32, 0, st>>>(
            in, static_cast<int>(n), K, m->W64[l]->as<double>(), m->b64[l]->as<double>(), out, st_i > 0 ? 1 : 0);
      } else {
        const dim3 grid(static_cast<unsigned>((N + 31) / 32), static_cast<unsigned>((n + 31) / 32));
        score_layer_kernel<<<grid, dim3(32, 8), 0, st>>>(
            in, rs, cs, static_cast<int>(n), K, m->W64[l]->as<double>(), m->b64[l]->as<double>(), out, N,
            last ? 0 : 1, last && st_i > 0 ? 1 : 0);
      }
      CUDA_OK(cudaGetLastError());
      in = out;
      rs = N;
      cs = 1;
    }
  }
}

felix_status felix_round(felix_space* s, const float* y, int64_t n, int32_t* sched, uint8_t* valid, void* stream) {
  FELIX_API_BEGIN
  if (!s || ((!y || !sched) && n > 0)) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL argument");
  if (n < 0 || n > (int64_t(1) << 30)) FELIX_THROW(FELIX_E_INVALID_ARG, "n out of range");
  if (n == 0) return FELIX_OK;
  DeviceGuard dg(s->device);
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  do_round(s, y, n, sched, st);
  if (valid) {
    ensure(s->phi64, static_cast<size_t>(n) * s->desc.froots.size() * 8);
    do_hard(s, sched, n, s->phi64.as<double>(), valid, st);
  }
  FELIX_API_END
}

felix_status felix_score(felix_space* s, felix_costmodel* m, const int32_t* sched, int64_t n, double* score, void* stream) {
  FELIX_API_BEGIN
  check_pair(s, m);
  if ((!sched || !score) && n > 0) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL argument");
  if (n < 0 || n > (int64_t(1) << 30)) FELIX_THROW(FELIX_E_INVALID_ARG, "n out of range");
  if (n == 0) return FELIX_OK;
  DeviceGuard dg(s->device);
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  ensure(s->phi64, static_cast<size_t>(n) * s->desc.froots.size() * 8);
  ensure(s->valid, static_cast<size_t>(n));
  do_hard(s, sched, n, s->phi64.as<double>(), s->valid.as<uint8_t>(), st);
  do_score(s, m, s->phi64.as<double>(), n, score, st);
  FELIX_API_END
}

felix_status felix_round_topk(felix_space* s, felix_costmodel* m, const float* y, int64_t n, int64_t index_base,
                              int32_t k, int64_t* idx_out, double* score_out, int32_t* sched_out, int32_t* n_out,
                              void* stream) {
  FELIX_API_BEGIN
  check_pair(s, m);
  if (!n_out || (k > 0 && (!idx_out || !score_out || !sched_out))) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL output");
  if (k < 0 || k > 1024) FELIX_THROW(FELIX_E_INVALID_ARG, "k must be in [0, 1024]");
  if (n < 0 || n > (int64_t(1) << 30) || (n > 0 && !y)) FELIX_THROW(FELIX_E_INVALID_ARG, "bad y / n");
  *n_out = 0;
  if (n == 0 || k == 0) return FELIX_OK;
  DeviceGuard dg(s->device);
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const int M = s->desc.n_vars;
  ensure(s->sched, static_cast<size_t>(n) * M * 4);
  ensure(s->valid, static_cast<size_t>(n));
  ensure(s->phi64, static_cast<size_t>(n) * s->desc.froots.size() * 8);
  ensure(s->score, static_cast<size_t>(n) * 8);
  do_round(s, y, n, s->sched.as<int32_t>(), st);
  do_hard(s, s->sched.as<int32_t>(), n, s->phi64.as<double>(), s->valid.as<uint8_t>(), st);
  do_score(s, m, s->phi64.as<double>(), n, s->score.as<double>(), st);
  ensure(s->fin_cand, static_cast<size_t>(k) * 4);
  // outputs packed in one device block and read back with a single copy into pinned memory:
  // [count (8 B) | idx k x 8 | score k x 8 | sched k x M x 4]
  const size_t pack_bytes = 8 + static_cast<size_t>(k) * 16 + static_cast<size_t>(k) * M * 4;
  ensure(s->o_pack, pack_bytes);
  if (s->h_pack_bytes < pack_bytes) {
    if (s->h_pack) cudaFreeHost(s->h_pack);
    s->h_pack = nullptr;
    s->h_pack_bytes = 0;
    CUDA_OK(cudaHostAlloc(&s->h_pack, pack_bytes, cudaHostAllocDefault));
    s->h_pack_bytes = pack_bytes;
  }
  uint8_t* pk = s->o_pack.as<uint8_t>();
  int* p_cnt = reinterpret_cast<int*>(pk);
  long long* p_idx = reinterpret_cast<long long*>(pk + 8);
  double* p_score = reinterpret_cast<double*>(pk + 8 + static_cast<size_t>(k) * 8);
  int32_t* p_sched = reinterpret_cast<int32_t*>(pk + 8 + static_cast<size_t>(k) * 16);
  run_topk(s, n, nullptr, s->sched.as<int32_t>(), M, k, s->fin_cand.as<int>(), p_cnt, st);
  topk_gather_kernel<<<1, std::max(32, (k + 31) / 32 * 32), 0, st>>>(
      s->fin_cand.as<int>(), p_cnt, k, s->score.as<double>(), s->sched.as<int32_t>(), M, index_base,
      p_idx, p_score, p_sched);
  CUDA_OK(cudaGetLastError());
  CUDA_OK(cudaMemcpyAsync(s->h_pack, pk, pack_bytes, cudaMemcpyDeviceToHost, st));
  CUDA_OK(cudaStreamSynchronize(st));
  const uint8_t* hp = static_cast<const uint8_t*>(s->h_pack);
  const int cnt = *reinterpret_cast<const int*>(hp);
  std::memcpy(idx_out, hp + 8, static_cast<size_t>(k) * 8);
  std::memcpy(score_out, hp + 8 + static_cast<size_t>(k) * 8, static_cast<size_t>(k) * 8);
  std::memcpy(sched_out, hp + 8 + static_cast<size_t>(k) * 16, static_cast<size_t>(k) * M * 4);
  *n_out = cnt;
  FELIX_API_END
}

felix_status felix_history_topk(felix_space* s, felix_costmodel* m, int32_t k, int64_t* idx_out, int32_t* step_out,
                                double* score_out, int32_t* sched_out, int32_t* n_out, int64_t* n_unique_out,
                                void* stream) {
  FELIX_API_BEGIN
  check_pair(s, m);
  if (!n_out || (k > 0 && (!idx_out || !step_out || !score_out || !sched_out))) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL output");
  if (k < 0 || k > 1024) FELIX_THROW(FELIX_E_INVALID_ARG, "k must be in [0, 1024]");
  if (!s->h_valid) FELIX_THROW(FELIX_E_INVALID_ARG, "the last felix_search did not record a history (history = 0)");
  *n_out = 0;
  DeviceGuard dg(s->device);
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const int M = s->desc.n_vars;
  int hc[2] = {0, 0};
  CUDA_OK(cudaMemcpyAsync(hc, s->h_cnt.p, 8, cudaMemcpyDeviceToHost, st));
  CUDA_OK(cudaStreamSynchronize(st));
  if (hc[1]) FELIX_THROW(FELIX_E_UNSUPPORTED, "history pool overflow");
  const int64_t n = std::min<int64_t>(hc[0], s->h_cap);
  if (n_unique_out) *n_unique_out = n;
  if (n == 0 || k == 0) return FELIX_OK;
  const int32_t* sched = s->h_pool_sched.as<int32_t>();
  ensure(s->valid, static_cast<size_t>(n));
  ensure(s->phi64, static_cast<size_t>(n) * s->desc.froots.size() * 8);
  ensure(s->score, static_cast<size_t>(n) * 8);
  do_hard(s, sched, n, s->phi64.as<double>(), s->valid.as<uint8_t>(), st);
  do_score(s, m, s->phi64.as<double>(), n, s->score.as<double>(), st);
  ensure(s->fin_cand, static_cast<size_t>(k) * 4);
  ensure(s->fin_cnt, 4);
  const long long* key = s->h_pool_key.as<long long>();
  run_topk(s, n, key, sched, M, k, s->fin_cand.as<int>(), s->fin_cnt.as<int>(), st);
  ensure(s->o_idx, static_cast<size_t>(k) * 8);
  ensure(s->o_step, static_cast<size_t>(k) * 4);
  ensure(s->o_score, static_cast<size_t>(k) * 8);
  ensure(s->o_sched, static_cast<size_t>(k) * M * 4);
  hist_gather_kernel<<<1, std::max(32, (k + 31) / 32 * 32), 0, st>>>(
      s->fin_cand.as<int>(), s->fin_cnt.as<int>(), k, s->score.as<double>(), sched, key, M, s->h_index_base,
      s->o_idx.as<long long>(), s->o_step.as<int>(), s->o_score.as<double>(), s->o_sched.as<int32_t>());
  CUDA_OK(cudaGetLastError());
  int cnt = 0;
  CUDA_OK(cudaMemcpyAsync(&cnt, s->fin_cnt.p, 4, cudaMemcpyDeviceToHost, st));
  CUDA_OK(cudaMemcpyAsync(idx_out, s->o_idx.p, static_cast<size_t>(k) * 8, cudaMemcpyDeviceToHost, st));
  CUDA_OK(cudaMemcpyAsync(step_out, s->o_step.p, static_cast<size_t>(k) * 4, cudaMemcpyDeviceToHost, st));
  CUDA_OK(cudaMemcpyAsync(score_out, s->o_score.p, static_cast<size_t>(k) * 8, cudaMemcpyDeviceToHost, st));
  CUDA_OK(cudaMemcpyAsync(sched_out, s->o_sched.p, static_cast<size_t>(k) * M * 4, cudaMemcpyDeviceToHost, st));
  CUDA_OK(cudaStreamSynchronize(st));
  *n_out = cnt;
  FELIX_API_END
}

felix_status felix_debug_trace(felix_space* s, uint64_t* out, int64_t n_words) {
  FELIX_API_BEGIN
  if (!s || !out) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL argument");
  DeviceGuard dg(s->device);
  // every kernel of a module is its own library with its own copy of the stamp arrays: read them all and
  // take the elementwise max (%globaltimer is monotonic; a kernel leaves the other kernels' slots at 0)
  auto read_max = [&](const felix_space::Module& m, const char* name, uint64_t* dst, size_t words) {
    bool found = false;
    std::vector<uint64_t> tmp(words);
    std::fill(dst, dst + words, uint64_t(0));
    for (cudaLibrary_t l : m.libs) {
      void* ptr = nullptr;
      size_t bytes = 0;
      if (!l || cudaLibraryGetGlobal(&ptr, &bytes, l, name) != cudaSuccess) { cudaGetLastError(); continue; }
      const size_t nw = std::min(words, bytes / 8);
      CUDA_OK(cudaMemcpy(tmp.data(), ptr, nw * 8, cudaMemcpyDeviceToHost));
      for (size_t i = 0; i < nw; ++i) dst[i] = std::max(dst[i], tmp[i]);
      found = true;
    }
    return found;
  };
  for (auto it = s->modules.rbegin(); it != s->modules.rend(); ++it) {   // widest P first (the search's)
    const size_t tw = std::min<size_t>(2 * 8192 * 8, static_cast<size_t>(n_words));
    if (!read_max(it->second, "felix_trace", out, tw)) continue;
    // then the per-warp cone-end stamps of the forward kernel, [8192][16], if the caller asked for them
    if (static_cast<size_t>(n_words) > tw)
      read_max(it->second, "felix_wtrace", out + tw, std::min<size_t>(8192 * 16, static_cast<size_t>(n_words) - tw));
    return FELIX_OK;
  }
  FELIX_THROW(FELIX_E_UNSUPPORTED, "no trace buffer (felix_tune(\"trace\", 1) before the kernels are generated)");
  FELIX_API_END
}

felix_status felix_tune(const char* key, int32_t value) {
  FELIX_API_BEGIN
  if (!key) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL key");
  const std::string k(key);
  auto in = [&](std::initializer_list<int> ok) {
    for (int v : ok) if (v == value) return;
    FELIX_THROW(FELIX_E_INVALID_ARG, "felix_tune: bad value " + std::to_string(value) + " for " + k);
  };
  if (k == "mlp") { in({-1, 0, 1, 2}); g_tune.mlp = value; }
  else if (k == "cone_width") { in({-1, 1, 2, 4, 8, 16}); g_tune.P = value; }
  else if (k == "replicas") { in({-1, 1, 2, 4}); g_tune.R = value; }
  else if (k == "sc_warps") { in({-1, 1, 2, 3, 4, 5, 6, 7, 8}); g_tune.scw = value; }
  else if (k == "chunks") { if (value != -1 && (value < 1 || value > 16)) in({}); g_tune.chunks = value; }
  else if (k == "split_cone") { in({-1, 0, 1}); g_tune.sc = value; }
  else if (k == "tile_cta_group") { in({-1, 1, 2}); g_tune.tile_cg = value; }
  else if (k == "chain_cta_group") { in({-1, 1, 2}); g_tune.chain_cg = value; }
  else if (k == "dphi_ksplit") { in({-1, 1, 2, 4}); g_tune.dphi_ksplit = value; }
  else if (k == "codegen_cone_width") { in({-1, 1, 2, 4, 8, 16}); g_tune.codegen_P = value; }
  else if (k == "codegen_replicas") { in({-1, 1, 2, 4}); g_tune.codegen_R = value; }
  else if (k == "trace") { in({0, 1}); g_tune.trace = value; }
  else if (k == "round_bnb") { in({0, 1}); g_tune.round_bnb = value; }
  else if (k == "score_dmma") { in({-1, 0, 1}); g_tune.score_dmma = value; }
  else if (k == "dphi_tma") { in({-1, 0, 1}); g_tune.dphi_tma = value; }
  else if (k == "pdl") { if (value != -1 && (value < 0 || value > 7)) in({}); g_tune.pdl = value; }
  else if (k == "graph_steps") { if (value != -1 && (value < 1 || value > 1000)) in({}); g_tune.graph_steps = value; }
  else FELIX_THROW(FELIX_E_INVALID_ARG, "felix_tune: unknown key " + k);
  FELIX_API_END
}

felix_status felix_profile_enable(felix_space* s, int32_t enable) {
  FELIX_API_BEGIN
  if (!s) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL space");
  s->profiling = enable != 0;
  FELIX_API_END
}

felix_status felix_profile_read(felix_space* s, double* ms, int64_t* launches) {
  FELIX_API_BEGIN
  if (!s || !ms || !launches) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL argument");
  DeviceGuard dg(s->device);
  for (auto& e : s->prof) {
    CUDA_OK(cudaEventSynchronize(e.b));
    float t = 0;
    CUDA_OK(cudaEventElapsedTime(&t, e.a, e.b));
    s->prof_ms[e.cls] += t;
    cudaEventDestroy(e.a);
    cudaEventDestroy(e.b);
  }
  s->prof.clear();
  for (int c = 0; c < 4; ++c) { ms[c] = s->prof_ms[c]; launches[c] = s->prof_launches[c]; }
  FELIX_API_END
}

felix_status felix_profile_reset(felix_space* s) {
  FELIX_API_BEGIN
  if (!s) FELIX_THROW(FELIX_E_INVALID_ARG, "NULL space");
  for (auto& e : s->prof) { cudaEventDestroy(e.a); cudaEventDestroy(e.b); }
  s->prof.clear();
  for (int c = 0; c < 4; ++c) { s->prof_ms[c] = 0; s->prof_launches[c] = 0; }
  FELIX_API_END
}

}  // extern "C"
