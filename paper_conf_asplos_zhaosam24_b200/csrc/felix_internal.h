// felix_internal.h — host-side structures of libfelix (not part of the ABI).
#pragma once
#include <cstdint>
#include <string>
#include <vector>
#include <memory>
#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include "../../include/felix.h"

namespace felix {

// -------------------------------------------------------------------------- errors
void set_error(const std::string& msg);
struct Error {
  felix_status code;
  std::string msg;
};
#define FELIX_THROW(code, msg) throw ::felix::Error{code, msg}
#define CUDA_OK(x)                                                                            \
  do {                                                                                        \
    cudaError_t e_ = (x);                                                                     \
    if (e_ != cudaSuccess)                                                                    \
      FELIX_THROW(e_ == cudaErrorMemoryAllocation ? FELIX_E_OOM : FELIX_E_CUDA,               \
                  std::string(#x) + ": " + cudaGetErrorString(e_));                           \
  } while (0)
#define CU_OK(x)                                                                              \
  do {                                                                                        \
    CUresult r_ = (x);                                                                        \
    if (r_ != CUDA_SUCCESS)                                                                   \
      FELIX_THROW(FELIX_E_CUDA, std::string(#x) + ": CUresult " + std::to_string((int)r_));   \
  } while (0)

// -------------------------------------------------------------------------- device buffers
struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
  DevBuf() = default;
  DevBuf(const DevBuf&) = delete;
  DevBuf& operator=(const DevBuf&) = delete;
  ~DevBuf() { if (p) cudaFree(p); }
  void alloc(size_t b) {
    if (p) { cudaFree(p); p = nullptr; }
    bytes = b;
    if (b) CUDA_OK(cudaMalloc(&p, b));
  }
  template <class T> T* as() const { return static_cast<T*>(p); }
};

// -------------------------------------------------------------------------- space description
struct SpaceDesc {
  int n_vars = 0;
  std::vector<felix_var> vars;
  std::vector<int64_t> split_extent;
  std::vector<std::vector<int32_t>> split_vars;
  std::vector<felix_node> nodes;
  std::vector<int32_t> froots, croots;
  int n_statements = 1;          // feature roots = n_statements per-statement vectors, statement-major
  int k0() const { return static_cast<int>(froots.size()) / n_statements; }
  int n_roots_total() const;
};

// split component tables for rounding (reading O10)
struct RoundTables {
  std::vector<int32_t> comp_nvars, comp_var0;     // per component: #vars, offset into comp_vars
  std::vector<int32_t> comp_vars;                 // concatenated var indices (ascending)
  std::vector<int64_t> comp_toff;                 // offset of the component's tuple block (in tuples)
  std::vector<int64_t> comp_tcount;
  std::vector<int64_t> comp_eoff;                 // offset (in elements) of its tuple entries
  std::vector<int32_t> tuples;                    // per tuple, |c| factors
  std::vector<double> lnf;                        // ln of each factor (host libm)
  std::vector<int32_t> int_vars;                  // INT variables
  std::vector<int64_t> int_lo, int_hi, int_toff;  // thresholds ln(k + 1/2), k in [lo, hi)
  std::vector<double> int_thr;
  int64_t n_tuples_total = 0;                     // rows of the tuple tables (components searched by scan)
  // branch-and-bound search (components with more than kRoundTableMax tuples, or all of them under
  // felix_tune("round_bnb", 1)): per component its splits, per component var its split mask and the
  // ascending divisors of the gcd of its splits' extents
  std::vector<int32_t> comp_ns, comp_s0;          // per component: #splits touching it, offset into comp_sext
  std::vector<int64_t> comp_sext;                 // extents of those splits
  std::vector<uint32_t> var_smask;                // per comp_vars entry: bit q <=> var is in the component's split q
  std::vector<int64_t> var_doff;                  // per comp_vars entry: offset of its divisor list
  std::vector<int32_t> var_dcnt;
  std::vector<int64_t> dval;                      // divisors (ascending) ...
  std::vector<double> dln;                        // ... and their ln (host libm, as the tables)
  std::vector<int32_t> bnb_comps;                 // components without a tuple table
};
constexpr int64_t kRoundTableMax = int64_t(1) << 16;   // larger components use the branch-and-bound kernel
constexpr int kRoundMaxSplits = 16;                      // splits touching one component (B&B register state)
void build_round_tables(const SpaceDesc& d, RoundTables& t);

// -------------------------------------------------------------------------- codegen
struct CodegenInfo {
  int64_t flops_fwd = 0;
  int64_t flops_rev = 0;
  int rev_smem_bytes = 0;
};
// P = warps cooperating on one 32-candidate block (cone partition of the roots), 1..8
std::string generate_dag_module(const SpaceDesc& d, int K0p, int P, int R, bool trace, int dphi_parts, CodegenInfo* info);

// -------------------------------------------------------------------------- cost model
struct CostModel {
  uint64_t uid = 0;              // process-wide unique id (workspace caches key on it, never on the address)
  int device = 0;
  int n_layers = 0;
  std::vector<int32_t> dims;     // dims[0..L]
  int K0p = 0;                   // dims[0] padded (GEMM K of layer 1, N of the dphi GEMM)
  // per layer l = 0..L-2 (weights W_{l+1} in paper numbering): forward (N x Kp) and transposed
  std::vector<std::unique_ptr<DevBuf>> W_hi, W_lo, WT_hi, WT_lo, bias;
  DevBuf head_w;                 // last layer row [dims[L-1]] fp32
  // first backward GEMM with the head row folded in: WTs[j][i] = -w_L[i] * W_{L-1}[i][j] (fp32 product, then
  // split), so its A operand is the exact 0/1 mask [Z_{L-1} > 0] (chain: no A lo pass, no A lo bytes)
  DevBuf WTs_hi, WTs_lo;
  float head_b = 0.f;
  std::vector<std::unique_ptr<DevBuf>> W64, b64;   // fp64 copies of every layer (scoring)
};

uint64_t next_uid();            // process-wide counter for CostModel / space identities

}  // namespace felix
