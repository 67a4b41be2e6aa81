// codegen.cpp — per-space straight-line CUDA for the feature-expression DAG, compiled with NVRTC.
//
// Felix's expression rewriter (Rust + egg, L1068-1071) turns feature formulas into
// smooth differentiable expressions, takes their logarithm and substitutes x = e^y.  Here the same
// rewrite is *emitted as code*: every DAG node is a named register value, the reverse sweep
// (Alg. 1 line 18) is straight-line adjoint code, fused with the loss / penalty seeds
// (Eq. 4) and the Adam update (L889-892).
//
// Work split ("cone partition"): the feature + constraint roots are partitioned into P groups of
// balanced cost; a CTA of P warps handles 32 candidates and warp g evaluates only the cone (the
// sub-DAG) of group g's roots — forward and reverse — for its 32 candidates.  Partial adjoints of
// x are summed across the P warps through shared memory in fixed order (deterministic).  This
// gives P-fold more, shorter dependency chains, so small populations (C2: 4096 candidates) fill
// the 148 SMs instead of one warp per SM.  Warp-uniform groups: no divergence.
//
// Generated kernels:
//   felix_fwd        smooth forward (FP64) -> phi = slog(F) as fp16 hi/lo rows (MMA A operand)
//   felix_rev_adam   recompute forward, seeds, reverse sweep, dL/dy, Adam
//   felix_rev_eval   same, writing phi / g / cost / loss / grad instead of updating y
//   felix_hard       hard semantics in FP64 (IEEE ops) at integer points -> slog features + validity
//   felix_init       rejection sampler (FP64 decisions, counter-based RNG)
//   felix_rev_sc     split-cone reverse (default search path): one cone per CTA, partial adjoints per cone
//   felix_fwd_adam   felix_fwd preceded by Adam step t-1 from those partials (in place)
//   felix_adam_sc    the last Adam step of a split-cone search
#include <algorithm>
#include <climits>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <functional>
#include <numeric>
#include <sstream>
#include <string>
#include <vector>
#include "felix_internal.h"

namespace felix {

namespace {

std::string lit(double v) {
  if (std::isinf(v)) return v > 0 ? "(1.0/0.0)" : "(-1.0/0.0)";
  char buf[64];
  snprintf(buf, sizeof buf, "%.17g", v);
  std::string s(buf);
  if (s.find_first_of(".eEn") == std::string::npos) s += ".0";
  return s;
}

const char* kPrelude = R"CUDA(
typedef unsigned long long u64;
typedef unsigned int u32;
typedef unsigned short u16;
__device__ __forceinline__ u16 f2h(float f) { u16 h; asm("cvt.rn.f16.f32 %0, %1;" : "=h"(h) : "f"(f)); return h; }
__device__ __forceinline__ float h2f(u16 h) { float f; asm("cvt.f32.f16 %0, %1;" : "=f"(f) : "h"(h)); return f; }
// ---- fast FP64 reciprocal / sqrt for the search kernels: MUFU seed + one Newton step (relative error
//      ~2^-44, far inside the 1e-4 feature tolerance; no slow path).  The hard / sampler kernels, which
//      take integer decisions, use IEEE '/' and sqrt.
__device__ __forceinline__ double f_rcp(double b) {
  double r0; asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r0) : "d"(b));
  const double e = fma(-b, r0, 1.0); const double r = fma(r0, e, r0);
  return (r0 == 0.0 || isinf(r0)) ? r0 : r;
}
// ---- FP32 helpers (MUFU approximations, ~2 ulp): the tails of the smooth step in the forward and the
//      whole split-cone reverse kernel (DESIGN.md "Precision of the expression kernels")
__device__ __forceinline__ float f_rcpf(float x) { float r; asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x)); return r; }
__device__ __forceinline__ float f_sqrtf(float x) { float r; asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x)); return r; }
__device__ __forceinline__ float sf_hyp(float t) { return f_sqrtf(fmaf(t, t, 1.f)); }
__device__ __forceinline__ float sf_tail(float t, float h) { return 0.5f * f_rcpf(h * (h + fabsf(t))); }
__device__ __forceinline__ float sf_Sh(float t, float h) { const float tl = sf_tail(t, h); return t >= 0.f ? 1.f - tl : tl; }
__device__ __forceinline__ float sf_dSh(float h) { return 0.5f * f_rcpf(h * h * h); }
__device__ __forceinline__ float sf_gaph(float t, float h) { return 0.5f * f_rcpf(h + fabsf(t)); }
// smooth step with an FP64 argument and an FP32 tail: t = a - b is exact in FP64 (no cancellation),
// the tail 1/(2h(h+|t|)) is only needed to relative precision (S = 1 - tail or tail in FP64)
__device__ __forceinline__ double sm_Sf(double t, float h) { const double tl = (double)sf_tail((float)t, h); return t >= 0.0 ? 1.0 - tl : tl; }
__device__ __forceinline__ float slogpf_(float f) { return f_rcpf((1.f + fabsf(f)) * 0.69314718055994530942f); }
__device__ __forceinline__ float f_powf(float a, float e) { return powf(a, e); }
__device__ __forceinline__ double f_div(double a, double b) { return a * f_rcp(b); }
__device__ __forceinline__ void cp_async4(float* dst, const float* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" :: "r"((unsigned)__cvta_generic_to_shared(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }
__device__ __forceinline__ double f_sqrt(double x) {
  double y; asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
  y = y * fma(-0.5 * x, y * y, 1.5);
  double s = x * y;
  s = fma(0.5 * y, fma(-s, s, x), s);
  return (x == 0.0 || isinf(x)) ? x : s;
}
// ---- smoothing kernel phi(t) = 1/2 (1+t^2)^(-3/2) (reading O3): S = step * phi, R = relu * phi
__device__ __forceinline__ double sm_hyp(double t) { return f_sqrt(fma(t, t, 1.0)); }
__device__ __forceinline__ double sm_S(double t) { const double h = sm_hyp(t); const double tail = 0.5 * f_rcp(h * (h + fabs(t))); return t >= 0.0 ? 1.0 - tail : tail; }
__device__ __forceinline__ double sm_dS(double t) { const double h = sm_hyp(t); return 0.5 * f_rcp(h * h * h); }
// variants taking h = sqrt(1+t^2) computed once by the forward and reused by the reverse sweep
__device__ __forceinline__ double sm_Sh(double t, double h) { const double tail = 0.5 * f_rcp(h * (h + fabs(t))); return t >= 0.0 ? 1.0 - tail : tail; }
__device__ __forceinline__ double sm_dSh(double h) { return 0.5 * f_rcp(h * h * h); }
__device__ __forceinline__ double sm_gaph(double t, double h) { return 0.5 * f_rcp(h + fabs(t)); }
// R(t) - relu(t) = 1/(2(sqrt(1+t^2) + |t|)); min / max without the cancellation of a - (a - b)
__device__ __forceinline__ double sm_gap(double t) { return 0.5 * f_rcp(sm_hyp(t) + fabs(t)); }
__device__ __forceinline__ double sm_min(double a, double b) { const double t = a - b; return (t >= 0.0 ? b : a) - sm_gap(t); }
__device__ __forceinline__ double sm_max(double a, double b) { const double t = a - b; return (t >= 0.0 ? a : b) + sm_gap(t); }
// IEEE versions for the integer-decision kernels
__device__ __forceinline__ double ie_hyp(double t) { double a = fabs(t); return a > 1.0 ? a * sqrt(1.0 + (1.0 / a) * (1.0 / a)) : sqrt(1.0 + t * t); }
__device__ __forceinline__ double ie_S(double t) { double h = ie_hyp(t); double tail = 1.0 / (2.0 * h * (h + fabs(t))); return t >= 0.0 ? 1.0 - tail : tail; }
__device__ __forceinline__ double ie_gap(double t) { return 1.0 / (2.0 * (ie_hyp(t) + fabs(t))); }
__device__ __forceinline__ double ie_min(double a, double b) { const double t = a - b; return (t >= 0.0 ? b : a) - ie_gap(t); }
__device__ __forceinline__ double ie_max(double a, double b) { const double t = a - b; return (t >= 0.0 ? a : b) + ie_gap(t); }
// slog(F) = sign(F) log2(1 + |F|)  (reading O4); fp32 suffices for the MMA operand
__device__ __forceinline__ float slogf_(double f) { float l = log2f(1.f + (float)fabs(f)); return f < 0.0 ? -l : l; }
__device__ __forceinline__ double slogp_(double f) { return f_rcp((1.0 + fabs(f)) * 0.69314718055994530942); }
__device__ __forceinline__ double slogd_(double f) { double l = log2(1.0 + fabs(f)); return f < 0.0 ? -l : (f > 0.0 ? l : 0.0); }
// counter-based uniform (include/felix.h felix_init_sample)
__device__ __forceinline__ u64 mix64(u64 z) { z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; return z ^ (z >> 31); }
__device__ __forceinline__ double cuni(u64 seed, u64 cand, u64 att, u64 var) {
  const u64 G = 0x9E3779B97F4A7C15ull;
  u64 h = seed;
  h = mix64(h + G * (cand + 1ull));
  h = mix64(h + G * (att + 1ull));
  h = mix64(h + G * (var + 1ull));
  return (double)(h >> 11) * (1.0 / 9007199254740992.0);
}
)CUDA";

int arity(int op) {
  switch (op) {
    case FELIX_OP_CONST: case FELIX_OP_VAR: return 0;
    case FELIX_OP_NEG: case FELIX_OP_EXP: case FELIX_OP_LOG: case FELIX_OP_SQRT: case FELIX_OP_NOT: case FELIX_OP_POW: return 1;
    case FELIX_OP_SELECT: return 3;
    default: return 2;
  }
}

// relative cost of a node in the search forward (FP64 values, FP32 smooth-step tails; SASS instructions of
// the emitted code, which is what the warps of a cone-group block wait on at their barrier): balances
// the cone partition.  A feature root adds kSlogCost (slog + shared-memory store).
int node_cost(int op) {
  switch (op) {
    case FELIX_OP_CONST: case FELIX_OP_VAR: return 0;
    case FELIX_OP_GT: case FELIX_OP_GE: case FELIX_OP_LT: case FELIX_OP_LE: return 12;
    case FELIX_OP_EQ: case FELIX_OP_NE: return 26;
    case FELIX_OP_MIN: case FELIX_OP_MAX: return 18;
    case FELIX_OP_DIV: case FELIX_OP_FLOORDIV: case FELIX_OP_CEILDIV: return 7;
    case FELIX_OP_SQRT: return 8;
    case FELIX_OP_EXP: case FELIX_OP_LOG: return 40;
    case FELIX_OP_POW: return 80;
    case FELIX_OP_SELECT: case FELIX_OP_OR: return 3;
    default: return 1;
  }
}
constexpr int kSlogCost = 10;

struct Gen {
  const SpaceDesc& d;
  int n;
  std::vector<bool> depvar;     // node depends on a variable
  std::ostringstream o;
  int64_t flops = 0;
  int64_t flops_rev = 0;   // arithmetic ops of the emitted reverse sweep (adjoint accumulations + local partials)

  std::vector<bool> isbool;     // comparison / logic node (FP32 mode keeps its complement c<i> = 1 - v<i>)

  explicit Gen(const SpaceDesc& dd) : d(dd), n((int)dd.nodes.size()), depvar(n, false), isbool(n, false) {
    for (int i = 0; i < n; ++i) {
      const int op_ = dd.nodes[i].op;
      isbool[i] = op_ == FELIX_OP_GT || op_ == FELIX_OP_GE || op_ == FELIX_OP_LT || op_ == FELIX_OP_LE || op_ == FELIX_OP_EQ ||
                  op_ == FELIX_OP_NE || op_ == FELIX_OP_AND || op_ == FELIX_OP_OR || op_ == FELIX_OP_NOT;
    }
    for (int i = 0; i < n; ++i) {
      const felix_node& nd = d.nodes[i];
      if (nd.op == FELIX_OP_VAR) { depvar[i] = true; continue; }
      if (nd.op == FELIX_OP_CONST) continue;
      const int ar = arity(nd.op);
      bool dv = false;
      if (ar >= 1) dv |= depvar[nd.a];
      if (ar >= 2) dv |= depvar[nd.b];
      if (ar >= 3) dv |= depvar[nd.c];
      depvar[i] = dv;
    }
  }

  std::vector<bool> cone(const std::vector<int>& roots) const {
    std::vector<bool> in(n, false);
    for (int r : roots) in[r] = true;
    for (int i = n - 1; i >= 0; --i) {
      if (!in[i]) continue;
      const felix_node& nd = d.nodes[i];
      const int ar = arity(nd.op);
      if (ar >= 1) in[nd.a] = true;
      if (ar >= 2) in[nd.b] = true;
      if (ar >= 3) in[nd.c] = true;
    }
    return in;
  }

  // forward node values for the nodes in `in`.  mode 0: search forward (FP64 values, FP32 tails of the
  // smooth step), 1: IEEE smooth FP64 (sampler), 2: hard FP64 (integer points), 3: FP32 (split-cone
  // reverse kernel).  Smooth compare / min / max nodes keep t and h = sqrt(1+t^2) as named values for
  // the reverse sweep: compares as FP32 hf<i> (and kf<i> for EQ/NE), min / max as h<i> in the node's type.
  // complement 1 - v of a BOOL operand in FP32 mode (a CONST used as a condition has none stored)
  std::string cmp_of(int j) const {
    return isbool[j] ? "c" + std::to_string(j) : "(1.f - v" + std::to_string(j) + ")";
  }

  // FP32 forward of the BOOL / SELECT nodes with complements: a smooth step near 1 keeps its tail in
  // c<i> (1 - S rounded to 1.f would lose it), and a SELECT uses the complement of its condition on the
  // side where the condition is near 1, so  select(c, a, b) = a + (b - a) (1 - c)  with (1 - c) exact to
  // FP32 relative precision (e.g. b = 5e9, 1 - c = 1.9e-8: the value 98 that b + (a - b) c loses in FP32).
  bool emit_f32_bool(int i, const char* ind) {
    const felix_node& nd = d.nodes[i];
    const std::string A = "v" + std::to_string(nd.a), B = "v" + std::to_string(nd.b), C = "v" + std::to_string(nd.c);
    const std::string I = std::to_string(i);
    switch (nd.op) {
      case FELIX_OP_GT: case FELIX_OP_GE: case FELIX_OP_LT: case FELIX_OP_LE: {
        const bool ab = nd.op == FELIX_OP_GT || nd.op == FELIX_OP_GE;
        o << ind << "const float t" << I << " = " << (ab ? A + " - " + B : B + " - " + A) << ";\n"
          << ind << "const float hf" << I << " = sf_hyp(t" << I << ");\n"
          << ind << "const float tl" << I << " = sf_tail(t" << I << ", hf" << I << ");\n"
          << ind << "const float v" << I << " = t" << I << " >= 0.f ? 1.f - tl" << I << " : tl" << I << ";\n"
          << ind << "const float c" << I << " = t" << I << " >= 0.f ? tl" << I << " : 1.f - tl" << I << ";\n";
        flops += 6;
        return true;
      }
      case FELIX_OP_EQ: case FELIX_OP_NE: {
        o << ind << "const float d" << I << " = " << A << " - " << B << ";\n"
          << ind << "const float t" << I << " = d" << I << " + 0.5f;\n"
          << ind << "const float u" << I << " = 0.5f - d" << I << ";\n"
          << ind << "const float hf" << I << " = sf_hyp(t" << I << ");\n"
          << ind << "const float kf" << I << " = sf_hyp(u" << I << ");\n"
          << ind << "const float ta" << I << " = sf_tail(t" << I << ", hf" << I << "), tb" << I << " = sf_tail(u" << I << ", kf" << I << ");\n"
          << ind << "const float pa" << I << " = t" << I << " >= 0.f ? 1.f - ta" << I << " : ta" << I << ";\n"
          << ind << "const float qa" << I << " = t" << I << " >= 0.f ? ta" << I << " : 1.f - ta" << I << ";\n"
          << ind << "const float pb" << I << " = u" << I << " >= 0.f ? 1.f - tb" << I << " : tb" << I << ";\n"
          << ind << "const float qb" << I << " = u" << I << " >= 0.f ? tb" << I << " : 1.f - tb" << I << ";\n"
          << ind << "const float e" << I << " = pa" << I << " * pb" << I << ";\n"
          << ind << "const float ce" << I << " = qa" << I << " + qb" << I << " - qa" << I << " * qb" << I << ";\n"
          << ind << "const float v" << I << " = " << (nd.op == FELIX_OP_EQ ? "e" : "ce") << I << ";\n"
          << ind << "const float c" << I << " = " << (nd.op == FELIX_OP_EQ ? "ce" : "e") << I << ";\n";
        flops += 16;
        return true;
      }
      case FELIX_OP_AND:
        o << ind << "const float v" << I << " = " << A << " * " << B << ";\n"
          << ind << "const float c" << I << " = " << cmp_of(nd.a) << " + " << cmp_of(nd.b) << " - " << cmp_of(nd.a) << " * " << cmp_of(nd.b) << ";\n";
        flops += 4;
        return true;
      case FELIX_OP_OR:
        o << ind << "const float v" << I << " = " << A << " + " << B << " - " << A << " * " << B << ";\n"
          << ind << "const float c" << I << " = " << cmp_of(nd.a) << " * " << cmp_of(nd.b) << ";\n";
        flops += 4;
        return true;
      case FELIX_OP_NOT:
        o << ind << "const float v" << I << " = " << cmp_of(nd.a) << ";\n"
          << ind << "const float c" << I << " = " << A << ";\n";
        return true;
      case FELIX_OP_SELECT:
        o << ind << "const float v" << I << " = " << A << " >= 0.5f ? " << B << " + (" << C << " - " << B << ") * " << cmp_of(nd.a)
          << " : " << C << " + (" << B << " - " << C << ") * " << A << ";\n";
        flops += 3;
        return true;
      default:
        return false;
    }
  }

  void emit_forward(const std::vector<bool>& in, int mode, const char* xname, const char* ind = "  ") {
    const bool hard = mode == 2, f32 = mode == 3;
    const std::string T = f32 ? "float" : "double";
    const std::string one = f32 ? "1.f" : "1.0", half = f32 ? "0.5f" : "0.5";
    const std::string mn = mode == 0 ? "sm_min" : "ie_min", mx = mode == 0 ? "sm_max" : "ie_max",
                      S = mode == 0 ? "sm_S" : "ie_S";
    auto divx = [&](const std::string& a, const std::string& b) {
      if (f32) return a + " * f_rcpf(" + b + ")";
      return mode == 0 ? "f_div(" + a + ", " + b + ")" : "(" + a + " / " + b + ")";
    };
    auto cst = [&](double v) { return f32 ? "(float)" + lit(v) : lit(v); };
    for (int i = 0; i < n; ++i) {
      if (!in[i]) continue;
      const felix_node& nd = d.nodes[i];
      const std::string A = "v" + std::to_string(nd.a), B = "v" + std::to_string(nd.b), C = "v" + std::to_string(nd.c);
      std::string e;
      const std::string I = std::to_string(i);
      if (f32 && emit_f32_bool(i, ind)) continue;
      if (mode == 0 || f32) {
        switch (nd.op) {
          case FELIX_OP_GT: case FELIX_OP_GE: case FELIX_OP_LT: case FELIX_OP_LE: {
            const bool ab = nd.op == FELIX_OP_GT || nd.op == FELIX_OP_GE;
            o << ind << "const " << T << " t" << I << " = " << (ab ? A + " - " + B : B + " - " + A) << ";\n"
              << ind << "const float hf" << I << " = sf_hyp((float)t" << I << ");\n"
              << ind << "const " << T << " v" << I << " = " << (f32 ? "sf_Sh" : "sm_Sf") << "(t" << I << ", hf" << I << ");\n";
            flops += 6;
            continue;
          }
          case FELIX_OP_MIN: case FELIX_OP_MAX: {
            const bool mx_ = nd.op == FELIX_OP_MAX;
            o << ind << "const " << T << " t" << I << " = " << A << " - " << B << ";\n"
              << ind << "const " << T << " h" << I << " = " << (f32 ? "sf_hyp" : "sm_hyp") << "(t" << I << ");\n"
              << ind << "const " << T << " v" << I << " = (t" << I << " >= 0 ? " << (mx_ ? A : B) << " : " << (mx_ ? B : A) << ") "
              << (mx_ ? "+" : "-") << (f32 ? " sf_gaph(t" : " sm_gaph(t") << I << ", h" << I << ");\n";
            flops += 6;
            continue;
          }
          case FELIX_OP_EQ: case FELIX_OP_NE: {
            o << ind << "const " << T << " t" << I << " = (" << A << " - " << B << ") + " << half << ";\n"
              << ind << "const " << T << " u" << I << " = " << half << " - (" << A << " - " << B << ");\n"
              << ind << "const float hf" << I << " = sf_hyp((float)t" << I << ");\n"
              << ind << "const float kf" << I << " = sf_hyp((float)u" << I << ");\n"
              << ind << "const " << T << " p" << I << " = " << (f32 ? "sf_Sh" : "sm_Sf") << "(t" << I << ", hf" << I << ");\n"
              << ind << "const " << T << " q" << I << " = " << (f32 ? "sf_Sh" : "sm_Sf") << "(u" << I << ", kf" << I << ");\n"
              << ind << "const " << T << " v" << I << " = " << (nd.op == FELIX_OP_EQ ? "" : one + " - ") << "p" << I << " * q" << I << ";\n";
            flops += 13;
            continue;
          }
          default: break;
        }
      }
      switch (nd.op) {
        case FELIX_OP_CONST: e = cst(nd.imm); break;
        case FELIX_OP_VAR: e = std::string(xname) + std::to_string((int)nd.imm); break;
        case FELIX_OP_ADD: e = A + " + " + B; ++flops; break;
        case FELIX_OP_SUB: e = A + " - " + B; ++flops; break;
        case FELIX_OP_MUL: e = A + " * " + B; ++flops; break;
        case FELIX_OP_DIV: e = divx(A, B); ++flops; break;
        case FELIX_OP_NEG: e = "-" + A; break;
        case FELIX_OP_POW: e = (f32 ? "f_powf(" : "pow(") + A + ", " + cst(nd.imm) + ")"; ++flops; break;
        case FELIX_OP_EXP: e = (f32 ? "expf(" : "exp(") + A + ")"; ++flops; break;
        case FELIX_OP_LOG: e = (f32 ? "logf(" : "log(") + A + ")"; ++flops; break;
        case FELIX_OP_SQRT: e = (f32 ? "f_sqrtf(" : mode == 0 ? "f_sqrt(" : "sqrt(") + A + ")"; ++flops; break;
        case FELIX_OP_MIN: e = hard ? "fmin(" + A + ", " + B + ")" : mn + "(" + A + ", " + B + ")"; flops += 6; break;
        case FELIX_OP_MAX: e = hard ? "fmax(" + A + ", " + B + ")" : mx + "(" + A + ", " + B + ")"; flops += 6; break;
        case FELIX_OP_GT: e = hard ? "(" + A + " > " + B + " ? 1.0 : 0.0)" : S + "(" + A + " - " + B + ")"; flops += 6; break;
        case FELIX_OP_GE: e = hard ? "(" + A + " >= " + B + " ? 1.0 : 0.0)" : S + "(" + A + " - " + B + ")"; flops += 6; break;
        case FELIX_OP_LT: e = hard ? "(" + A + " < " + B + " ? 1.0 : 0.0)" : S + "(" + B + " - " + A + ")"; flops += 6; break;
        case FELIX_OP_LE: e = hard ? "(" + A + " <= " + B + " ? 1.0 : 0.0)" : S + "(" + B + " - " + A + ")"; flops += 6; break;
        case FELIX_OP_EQ: e = hard ? "(" + A + " == " + B + " ? 1.0 : 0.0)"
                                   : S + "((" + A + " - " + B + ") + 0.5) * " + S + "(0.5 - (" + A + " - " + B + "))"; flops += 12; break;
        case FELIX_OP_NE: e = hard ? "(" + A + " != " + B + " ? 1.0 : 0.0)"
                                   : "1.0 - " + S + "((" + A + " - " + B + ") + 0.5) * " + S + "(0.5 - (" + A + " - " + B + "))"; flops += 13; break;
        case FELIX_OP_AND: e = A + " * " + B; ++flops; break;
        case FELIX_OP_OR: e = A + " + " + B + " - " + A + " * " + B; flops += 3; break;
        case FELIX_OP_NOT: e = one + " - " + A; ++flops; break;
        case FELIX_OP_SELECT: e = hard ? "(" + A + " != 0.0 ? " + B + " : " + C + ")" : C + " + (" + B + " - " + C + ") * " + A; flops += 3; break;
        case FELIX_OP_FLOORDIV: e = hard ? "floor(" + A + " / " + B + ")" : divx(A, B); ++flops; break;
        case FELIX_OP_CEILDIV: e = hard ? "ceil(" + A + " / " + B + ")" : divx(A, B); ++flops; break;
        default: e = f32 ? "0.f" : "0.0"; break;
      }
      o << ind << "const " << T << " v" << i << " = " << e << ";\n";
    }
  }

  std::string adj(int node) const {
    return d.nodes[node].op == FELIX_OP_VAR ? "gx" + std::to_string((int)d.nodes[node].imm) : "a" + std::to_string(node);
  }

  // nodes that receive an adjoint from `roots` inside cone `in`
  std::vector<bool> rev_live(const std::vector<bool>& in, const std::vector<int>& roots) const {
    std::vector<bool> need(n, false);
    for (int r : roots) if (depvar[r]) need[r] = true;
    for (int i = n - 1; i >= 0; --i) {
      if (!need[i] || !in[i]) continue;
      const felix_node& nd = d.nodes[i];
      if (nd.op == FELIX_OP_VAR || nd.op == FELIX_OP_CONST) continue;
      const int ar = arity(nd.op);
      if (ar >= 1 && depvar[nd.a]) need[nd.a] = true;
      if (ar >= 2 && depvar[nd.b]) need[nd.b] = true;
      if (ar >= 3 && depvar[nd.c]) need[nd.c] = true;
    }
    return need;
  }

  void emit_adj_decls(const std::vector<bool>& need, const char* ind, bool f32) {
    for (int i = 0; i < n; ++i)
      if (need[i] && d.nodes[i].op != FELIX_OP_VAR) o << ind << (f32 ? "float" : "double") << " a" << i << " = 0;\n";
  }

  // Reverse sweep over the values of emit_forward (mode 0 -> FP64 adjoints, mode 3 -> FP32 adjoints):
  // every local partial derivative is evaluated from the forward values and multiplies the adjoint.
  void emit_reverse_body(const std::vector<bool>& need, const char* ind, bool f32 = false) {
    const std::string T = f32 ? "float" : "double", one = f32 ? "1.f" : "1.0";
    auto acc = [&](int tgt, const std::string& expr, bool neg = false) {
      if (!depvar[tgt]) return;
      o << ind << "  " << adj(tgt) << (neg ? " -= " : " += ") << expr << ";\n";
    };
    auto J = [&](const std::string& e) { return "(" + T + ")(" + e + ")"; };
    const std::string rcp = f32 ? "f_rcpf(" : "f_rcp(";
    for (int i = n - 1; i >= 0; --i) {
      const felix_node& nd = d.nodes[i];
      if (!need[i] || nd.op == FELIX_OP_VAR || nd.op == FELIX_OP_CONST) continue;
      const std::string g = "a" + std::to_string(i);
      const std::string A = "v" + std::to_string(nd.a), B = "v" + std::to_string(nd.b), C = "v" + std::to_string(nd.c);
      const std::string V = "v" + std::to_string(i);
      const std::string I = std::to_string(i);
      o << ind << "{\n";
      switch (nd.op) {
        case FELIX_OP_ADD: case FELIX_OP_SUB: flops_rev += 2; break;
        case FELIX_OP_NEG: case FELIX_OP_NOT: flops_rev += 1; break;
        case FELIX_OP_MUL: case FELIX_OP_AND: flops_rev += 4; break;
        case FELIX_OP_DIV: case FELIX_OP_FLOORDIV: case FELIX_OP_CEILDIV: flops_rev += 6; break;
        case FELIX_OP_POW: flops_rev += 5; break;
        case FELIX_OP_EXP: flops_rev += 2; break;
        case FELIX_OP_LOG: case FELIX_OP_SQRT: flops_rev += 4; break;
        case FELIX_OP_MIN: case FELIX_OP_MAX: flops_rev += 9; break;
        case FELIX_OP_GT: case FELIX_OP_GE: case FELIX_OP_LT: case FELIX_OP_LE: flops_rev += 8; break;
        case FELIX_OP_EQ: case FELIX_OP_NE: flops_rev += 16; break;
        case FELIX_OP_OR: flops_rev += 6; break;
        case FELIX_OP_SELECT: flops_rev += 7; break;
        default: break;
      }
      switch (nd.op) {
        case FELIX_OP_ADD: acc(nd.a, g); acc(nd.b, g); break;
        case FELIX_OP_SUB: acc(nd.a, g); acc(nd.b, g, true); break;
        case FELIX_OP_MUL: acc(nd.a, g + " * " + J(B)); acc(nd.b, g + " * " + J(A)); break;
        case FELIX_OP_DIV: case FELIX_OP_FLOORDIV: case FELIX_OP_CEILDIV:
          o << ind << "  const " << T << " t = " << g << " * " << J(rcp + B + ")") << ";\n";
          acc(nd.a, "t"); acc(nd.b, "t * " + J(V), true); break;
        case FELIX_OP_NEG: acc(nd.a, g, true); break;
        case FELIX_OP_POW:
          acc(nd.a, g + " * " + J(f32 ? "(float)" + lit(nd.imm) + " * f_powf(" + A + ", (float)" + lit(nd.imm - 1.0) + ")"
                                       : lit(nd.imm) + " * pow(" + A + ", " + lit(nd.imm - 1.0) + ")")); break;
        case FELIX_OP_EXP: acc(nd.a, g + " * " + J(V)); break;
        case FELIX_OP_LOG: acc(nd.a, g + " * " + J(rcp + A + ")")); break;
        case FELIX_OP_SQRT: acc(nd.a, g + " * " + J((f32 ? "0.5f * " : "0.5 * ") + rcp + V + ")")); break;
        case FELIX_OP_MAX: case FELIX_OP_MIN:
          if (f32) {   // S(t) and 1 - S(t) both from the tail
            o << ind << "  const float tl = sf_tail(t" << I << ", h" << I << ");\n"
              << ind << "  const float s = t" << I << " >= 0.f ? 1.f - tl : tl, cs = t" << I << " >= 0.f ? tl : 1.f - tl;\n";
          } else {
            o << ind << "  const double s = sm_Sh(t" << I << ", h" << I << "), cs = 1.0 - s;\n";
          }
          if (nd.op == FELIX_OP_MAX) { acc(nd.a, g + " * s"); acc(nd.b, g + " * cs"); }
          else { acc(nd.a, g + " * cs"); acc(nd.b, g + " * s"); }
          break;
        case FELIX_OP_GT: case FELIX_OP_GE:
          o << ind << "  const " << T << " t = " << g << " * " << J("sf_dSh(hf" + I + ")") << ";\n";
          acc(nd.a, "t"); acc(nd.b, "t", true); break;
        case FELIX_OP_LT: case FELIX_OP_LE:
          o << ind << "  const " << T << " t = " << g << " * " << J("sf_dSh(hf" + I + ")") << ";\n";
          acc(nd.a, "t", true); acc(nd.b, "t"); break;
        case FELIX_OP_EQ: case FELIX_OP_NE: {
          if (f32) {
            // d/dd [S(d+1/2) S(1/2-d)] without the cancellation of S'(a) S(b) - S(a) S'(b) near d = 0:
            // -d/2 [(ha^2 + ha hb + hb^2)/(ha + hb) + 1 + a^2 + ab + b^2] / (ha^3 hb^3), a = d+1/2, b = 1/2-d
            o << ind << "  const float ha = hf" << I << ", hb = kf" << I << ", a_ = t" << I << ", b_ = u" << I << ";\n"
              << ind << "  const float der = -0.5f * d" << I << " * ((ha * ha + ha * hb + hb * hb) * f_rcpf(ha + hb) + 1.f + a_ * a_ + a_ * b_ + b_ * b_)"
              << " * f_rcpf(ha * ha * ha * hb * hb * hb);\n"
              << ind << "  const float t = " << (nd.op == FELIX_OP_EQ ? "" : "-") << g << " * der;\n";
          } else {
            o << ind << "  const double t = " << (nd.op == FELIX_OP_EQ ? "" : "-") << g << " * "
              << "((double)sf_dSh(hf" << I << ") * q" << I << " - p" << I << " * (double)sf_dSh(kf" << I << "));\n";
          }
          acc(nd.a, "t"); acc(nd.b, "t", true); break;
        }
        case FELIX_OP_AND: acc(nd.a, g + " * " + J(B)); acc(nd.b, g + " * " + J(A)); break;
        case FELIX_OP_OR:
          if (f32) { acc(nd.a, g + " * " + cmp_of(nd.b)); acc(nd.b, g + " * " + cmp_of(nd.a)); }
          else { acc(nd.a, g + " * " + J(one + " - " + B)); acc(nd.b, g + " * " + J(one + " - " + A)); }
          break;
        case FELIX_OP_NOT: acc(nd.a, g, true); break;
        case FELIX_OP_SELECT:
          acc(nd.a, g + " * " + J(B + " - " + C)); acc(nd.b, g + " * " + J(A));
          acc(nd.c, g + " * " + (f32 ? cmp_of(nd.a) : J(one + " - " + A))); break;
        default: break;
      }
      o << ind << "}\n";
    }
  }
};

// greedy partition of the roots into P groups of balanced cone cost
struct Partition {
  std::vector<std::vector<int>> feat;   // feature indices k per group
  std::vector<std::vector<int>> cons;   // user constraint indices r per group
};

Partition partition_roots(const Gen& g, const SpaceDesc& d, int P) {
  const int K = (int)d.froots.size(), Ru = (int)d.croots.size();
  struct Item { bool is_feat; int idx; int node; int64_t cost; };
  std::vector<Item> items;
  auto cone_cost = [&](int node) {
    auto c = g.cone({node});
    int64_t cost = 0;
    for (int i = 0; i < g.n; ++i) if (c[i]) cost += node_cost(d.nodes[i].op);
    return cost;
  };
  for (int k = 0; k < K; ++k) {
    const int r = d.froots[k];
    if (!g.depvar[r]) continue;      // constant features: group 0 writes them, no compute
    items.push_back({true, k, r, cone_cost(r) + kSlogCost});
  }
  for (int r = 0; r < Ru; ++r) items.push_back({false, r, d.croots[r], cone_cost(d.croots[r])});
  std::stable_sort(items.begin(), items.end(), [](const Item& a, const Item& b) { return a.cost > b.cost; });
  Partition part;
  part.feat.assign(P, {});
  part.cons.assign(P, {});
  std::vector<std::vector<bool>> in(P, std::vector<bool>(g.n, false));
  std::vector<int64_t> gcost(P, 0);
  for (const auto& it : items) {
    auto c = g.cone({it.node});
    int best = 0;
    int64_t best_total = INT64_MAX;
    for (int q = 0; q < P; ++q) {
      int64_t add = it.is_feat ? kSlogCost : 0;
      for (int i = 0; i < g.n; ++i) if (c[i] && !in[q][i]) add += node_cost(d.nodes[i].op);
      if (gcost[q] + add < best_total) { best_total = gcost[q] + add; best = q; }
    }
    for (int i = 0; i < g.n; ++i) if (c[i]) in[best][i] = true;
    gcost[best] = best_total;
    (it.is_feat ? part.feat : part.cons)[best].push_back(it.idx);
  }
  for (auto& v : part.feat) std::sort(v.begin(), v.end());
  for (auto& v : part.cons) std::sort(v.begin(), v.end());
  return part;
}

}  // namespace

int SpaceDesc::n_roots_total() const {
  int n_split = 0, n_int = 0;
  for (const auto& v : vars) (v.kind == FELIX_VAR_SPLIT ? n_split : n_int)++;
  return (int)croots.size() + n_split + (int)split_extent.size() + 2 * n_int;
}

std::string generate_dag_module(const SpaceDesc& d, int K0p, int P, int NREPv, bool trace, int dphi_parts, CodegenInfo* info) {
  Gen g(d);
  // dL/dphi of feature row `idx`, summed over the MLP's split-K partial slabs in fixed order (compile-time
  // unrolled: a runtime loop per seed makes NVRTC 3.5x slower on these straight-line kernels)
  auto dphi_at = [&](const std::string& idx) {
    std::string e = "dphi[" + idx + "]";
    for (int pp = 1; pp < dphi_parts; ++pp) e = "(" + e + " + dphi[" + idx + " + (size_t)" + std::to_string(pp) + " * K0P * ld_dphi])";
    return e;
  };
  std::ostringstream& o = g.o;
  const int M = d.n_vars, K = (int)d.froots.size(), Ru = (int)d.croots.size();
  const int R = d.n_roots_total(), Ra = R - Ru;
  const int NS = d.n_statements, K0 = K / NS;   // per-statement feature vectors (TenSet segment sum)
  // feature k -> (statement, index within the statement's vector)
  auto fs = [&](int k) { return k / K0; };
  auto fk = [&](int k) { return k % K0; };
  if (NREPv < 1) NREPv = 1;
  o << kPrelude;

  if (trace)
    o << "__device__ unsigned long long felix_trace[2][8192][8];\n"
         "__device__ unsigned long long felix_wtrace[8192][16];\n"
         "#define TWSTAMP() do { if ((threadIdx.x & 31) == 0 && blockIdx.x < 8192 && (threadIdx.x >> 5) < 16) { unsigned long long t_; asm volatile(\"mov.u64 %0, %globaltimer;\" : \"=l\"(t_)); felix_wtrace[blockIdx.x][threadIdx.x >> 5] = t_; } } while (0)\n"
         "#define TSTAMP(k, s) do { if (threadIdx.x == 0 && blockIdx.x < 8192) { unsigned long long t_; asm volatile(\"mov.u64 %0, %globaltimer;\" : \"=l\"(t_)); felix_trace[k][blockIdx.x][s] = t_; } } while (0)\n";
  else
    o << "#define TSTAMP(k, s) do {} while (0)\n#define TWSTAMP() do {} while (0)\n";
  o << "#define NV " << M << "\n#define NF " << K << "\n#define NRU " << Ru << "\n#define NR " << R
    << "\n#define NRA " << Ra << "\n#define K0P " << K0p << "\n#define PG " << P << "\n#define NS " << NS
    << "\n#define NREP " << NREPv << "\n";

  // ---------------------------------------------------------------- automatic validity roots (y space)
  struct Auto { std::string val; std::vector<std::pair<int, int>> terms; };
  std::vector<Auto> autos;
  for (int j = 0; j < M; ++j)
    if (d.vars[j].kind == FELIX_VAR_SPLIT) autos.push_back({"-y" + std::to_string(j), {{j, -1}}});
  for (size_t s = 0; s < d.split_extent.size(); ++s) {
    std::string e = "(";
    std::vector<std::pair<int, int>> t;
    for (size_t k = 0; k < d.split_vars[s].size(); ++k) {
      const int j = d.split_vars[s][k];
      e += (k ? " + y" : "y") + std::to_string(j);
      t.push_back({j, +1});
    }
    e += ") - " + lit(std::log((double)d.split_extent[s]));
    autos.push_back({e, t});
  }
  for (int j = 0; j < M; ++j)
    if (d.vars[j].kind == FELIX_VAR_INT) {
      autos.push_back({lit(std::log((double)d.vars[j].lo)) + " - y" + std::to_string(j), {{j, -1}}});
      autos.push_back({"y" + std::to_string(j) + " - " + lit(std::log((double)d.vars[j].hi)), {{j, +1}}});
    }

  const Partition part = partition_roots(g, d, P);
  std::vector<std::vector<bool>> fcone(P), rcone(P);
  std::vector<std::vector<int>> froots_g(P), rroots_g(P);
  for (int q = 0; q < P; ++q) {
    for (int k : part.feat[q]) froots_g[q].push_back(d.froots[k]);
    rroots_g[q] = froots_g[q];
    for (int r : part.cons[q]) rroots_g[q].push_back(d.croots[r]);
    fcone[q] = g.cone(froots_g[q]);
    rcone[q] = g.cone(rroots_g[q]);
  }
  auto vars_in = [&](const std::vector<bool>& c) {
    std::vector<bool> used(M, false);
    for (int i = 0; i < g.n; ++i)
      if (c[i] && d.nodes[i].op == FELIX_OP_VAR) used[(int)d.nodes[i].imm] = true;
    return used;
  };
  // arithmetic ops of one full forward evaluation (reported by felix_space_info)
  int64_t flops_fwd = 0, flops_rev = 0;
  {
    std::ostringstream save;
    save << o.str();
    std::vector<bool> all(g.n, true);
    g.flops = 0;
    g.emit_forward(all, 0, "x");
    flops_fwd = g.flops;
    std::vector<int> allroots(d.froots.begin(), d.froots.end());
    allroots.insert(allroots.end(), d.croots.begin(), d.croots.end());
    g.flops_rev = 0;
    g.emit_reverse_body(g.rev_live(all, allroots), "");
    flops_rev = g.flops_rev;
    o.str("");
    o.clear();
    o << save.str();
  }

  // ---------------------------------------------------------------- felix_fwd
  // block = PG warps x 32 candidates; warp q evaluates the features of group q; rows are staged in
  // shared memory and written out as contiguous 16-byte stores.  With NS statements, statement s of
  // candidate c is MLP row s * n + c.
  // NREP replicas of the PG groups per block, each on its own 32 candidates: warps running the same
  // cone's straight-line code share the SM's instruction fetches (the code is executed once per warp).
  // ADAM = 1 (felix_fwd_adam, split-cone searches): first apply Adam step s = *step_ctr - 1 (the reverse
  // kernel of the previous step left its partial adjoints in part / pen) to this CTA's 32 candidates in
  // place -- thread (wq, lane) owns vars j = wq + PG * jj, every load is issued before the first use --
  // then evaluate the features at the new y.  Each CTA owns its candidates, so in-place is race-free.
  // The arithmetic and its order are those of rev_body (sums over q = 0..P-1, seeds, Adam expression).
  auto emit_autos = [&](const char* ind, const std::string& ysrc) {
    for (int j = 0; j < M; ++j) o << ind << "const double y" << j << " = (double)" << ysrc << "[" << j << "]" << (ysrc == "sy" ? "[lane]" : "") << ";\n";
    for (size_t q = 0; q < autos.size(); ++q) o << ind << "const double spa" << q << " = fmax(" << autos[q].val << ", 0.0);\n";
    for (size_t q = 0; q < autos.size(); ++q) o << ind << "pen_ += spa" << q << " * spa" << q << ";\n";
  };
  auto emit_auto_grad_switch = [&](const char* ind) {
    o << ind << "switch (j) {\n";
    for (int j = 0; j < M; ++j) {
      std::string terms;
      for (size_t q = 0; q < autos.size(); ++q)
        for (auto& tv : autos[q].terms)
          if (tv.first == j) terms += std::string(tv.second > 0 ? " + " : " - ") + "spa" + std::to_string(q);
      if (!terms.empty()) o << ind << "  case " << j << ": gd += 2.0 * dlam * (0.0" << terms << "); break;\n";
    }
    o << ind << "  default: break;\n" << ind << "}\n";
  };
  // the automatic-root terms of dL/dy_j computed inside var j's case (felix_fwd_adam: a thread needs only
  // the autos of its own vars; the loss itself is not formed there, only its finiteness matters)
  auto emit_auto_grad_switch_inline = [&](const char* ind) {
    o << ind << "switch (j) {\n";
    for (int j = 0; j < M; ++j) {
      std::string terms;
      for (size_t q = 0; q < autos.size(); ++q)
        for (auto& tv : autos[q].terms)
          if (tv.first == j) terms += std::string(tv.second > 0 ? " + " : " - ") + "fmax(" + autos[q].val + ", 0.0)";
      if (!terms.empty()) o << ind << "  case " << j << ": gd += 2.0 * dlam * (0.0" << terms << "); break;\n";
    }
    o << ind << "  default: break;\n" << ind << "}\n";
  };
  o << "template <int ADAM>\n__device__ __forceinline__ void fwd_body(float* yv, int n, int ldy, u16* __restrict__ phi_hi, u16* __restrict__ phi_lo, int* step_ctr,\n"
    << "    float* mv, float* vv, const float* __restrict__ part, const double* __restrict__ pen, const float* __restrict__ c_part,\n"
    << "    int n_head_tiles, int ld_c, float head_b, float lam, float lr, float b1, float b2, float eps) {\n"
    << "  __shared__ float sphi_all[NREP][NS][32][K0P + 1];\n"
    << "  __shared__ double sx_all[NREP][NV][32];   // x = exp(y), computed once per replica and shared by its groups\n"
    << "  const int rep = threadIdx.x / (PG * 32), tid = threadIdx.x % (PG * 32);\n"
    << "  float (&sphi)[NS][32][K0P + 1] = sphi_all[rep];\n"
    << "  double (&sx)[NV][32] = sx_all[rep];\n"
    << "  const int lane = threadIdx.x & 31, wq = tid >> 5;\n"
    << "  const int c0 = (blockIdx.x * NREP + rep) * 32;\n"
    << "  asm volatile(\"griddepcontrol.launch_dependents;\" ::: \"memory\");\n"
    << "  TSTAMP(0, 0);\n"
    << "  asm volatile(\"griddepcontrol.wait;\" ::: \"memory\");   // y is the previous step's output\n"
    << "  TSTAMP(0, 1);\n"
    << "  if (!ADAM) {\n"
    << "    if (blockIdx.x == 0 && threadIdx.x == 0 && step_ctr) *step_ctr += 1;\n"
    << "    for (int e = tid; e < NV * 32; e += PG * 32) { const int l = e & 31; const int cl = c0 + l; sx[e >> 5][l] = exp((double)yv[(size_t)(e >> 5) * ldy + (cl < n ? cl : n - 1)]); }\n"
    << "  } else {\n"
    << "    __shared__ float sya_all[NREP][NV][32];\n"
    << "    __shared__ unsigned sbad_all[NREP][PG];\n"
    << "    float (&sy)[NV][32] = sya_all[rep];\n    unsigned* sbad = sbad_all[rep];\n"
    << "    constexpr int NJ = (NV + PG - 1) / PG;\n"
    << "    const int cl = c0 + lane;\n    const bool live = cl < n;\n    const int cc = live ? cl : n - 1;\n"
    << "    float yl[NJ], ml[NJ], vl[NJ], gxa[NJ];\n"
    << "#pragma unroll\n    for (int jj = 0; jj < NJ; ++jj) {\n"
    << "      const int j = wq + PG * jj;\n      if (j >= NV) break;\n"
    << "      yl[jj] = yv[(size_t)j * ldy + cc]; ml[jj] = mv[(size_t)j * n + cc]; vl[jj] = vv[(size_t)j * n + cc];\n"
    << "      float a = 0.f;\n#pragma unroll\n      for (int q = 0; q < PG; ++q) a += part[((size_t)q * NV + j) * n + cc];\n"
    << "      gxa[jj] = a;\n    }\n"
    // the loss inputs are requested with the rest (one memory round trip before the first barrier)
    << "    double pen_ = 0.0;\n"
    << "#pragma unroll\n    for (int q = 0; q < PG; ++q) pen_ += pen[(size_t)q * n + cc];\n"
    << "    float cst = head_b * NS;\n"
    << "#pragma unroll 4\n    for (int i = 0; i < NS * n_head_tiles; ++i) cst += c_part[(size_t)(i % n_head_tiles) * ld_c + (size_t)(i / n_head_tiles) * n + cc];\n"
    << "    const int s_ = *step_ctr - 1;   // Adam steps to apply: reverse kernels run so far (the counter starts at 1)\n"
    << "#pragma unroll\n    for (int jj = 0; jj < NJ; ++jj) { const int j = wq + PG * jj; if (j >= NV) break; sy[j][lane] = yl[jj]; }\n"
    << "    __syncthreads();\n    TSTAMP(0, 5);\n"
    << "    if (s_ <= 0) {\n"
    << "#pragma unroll\n      for (int jj = 0; jj < NJ; ++jj) { const int j = wq + PG * jj; if (j >= NV) break; sx[j][lane] = exp((double)yl[jj]); }\n"
    << "    } else {\n"
    << "      const double dlam = (double)lam;\n"
    // bias corrections first: independent of the loads and the barrier below, so they overlap them
    << "      const float bc1 = 1.f - powf(b1, (float)s_), bc2 = 1.f - powf(b2, (float)s_);\n"
    << "      const float step = lr / bc1, rb = 1.f / sqrtf(bc2);\n";
  // the loss -C + lam (user penalties + auto penalties) is finite iff C and the user penalties are (the
  // auto penalties are finite for finite y; a non-finite y makes its own gradient non-finite)
  for (int j = 0; j < M; ++j) o << "      const double y" << j << " = (double)sy[" << j << "][lane];\n";
  o << "      bool ok = isfinite(cst) && isfinite(pen_);\n"
    << "      float gyv[NJ];\n"
    << "#pragma unroll\n      for (int jj = 0; jj < NJ; ++jj) {\n"
    << "        const int j = wq + PG * jj;\n        if (j >= NV) break;\n"
    << "        double gd = (double)gxa[jj];   // the partials are dL/dy already (x_j folded in by felix_rev_sc)\n";
  emit_auto_grad_switch_inline("        ");
  o << "        gyv[jj] = (float)gd;\n        ok = ok && isfinite(gyv[jj]);\n      }\n"
    << "      const unsigned bad = __ballot_sync(0xffffffffu, !ok);\n"
    << "      if (lane == 0) sbad[wq] = bad;\n"
    << "      __syncthreads();\n      TSTAMP(0, 6);\n"
    << "      unsigned anybad = 0;\n#pragma unroll\n      for (int q = 0; q < PG; ++q) anybad |= sbad[q];\n"
    << "      const bool okall = !((anybad >> lane) & 1u);\n"
    << "#pragma unroll\n      for (int jj = 0; jj < NJ; ++jj) {\n"
    << "        const int j = wq + PG * jj;\n        if (j >= NV) break;\n"
    << "        float yy = yl[jj];\n"
    << "        if (okall) {\n"
    << "          float m = ml[jj], v = vl[jj];\n"
    << "          m = b1 * m + (1.f - b1) * gyv[jj]; v = b2 * v + (1.f - b2) * gyv[jj] * gyv[jj];\n"
    << "          yy = yl[jj] - step * m / (sqrtf(v) * rb + eps);\n"
    << "          if (live) { mv[(size_t)j * n + cl] = m; vv[(size_t)j * n + cl] = v; yv[(size_t)j * ldy + cl] = yy; }\n"
    << "        }\n"
    << "        sx[j][lane] = exp((double)yy);\n      }\n"
    << "    }\n  }\n"
    << "  TSTAMP(0, 7);\n  for (int k = tid; k < NS * 32 * (K0P + 1); k += PG * 32) (&sphi[0][0][0])[k] = 0.f;\n"
    << "  __syncthreads();\n  TSTAMP(0, 2);\n";
  for (int q = 0; q < P; ++q) {
    o << "  if (wq == " << q << ") {\n";
    if (q == 0)
      for (int k = 0; k < K; ++k)
        if (!g.depvar[d.froots[k]]) {
          // constant feature: value of its (var-free) cone, evaluated here
          o << "    {\n";
          g.emit_forward(g.cone({d.froots[k]}), 0, "x", "      ");
          o << "      sphi[" << fs(k) << "][lane][" << fk(k) << "] = slogf_(v" << d.froots[k] << ");\n    }\n";
        }
    const auto used = vars_in(fcone[q]);
    for (int j = 0; j < M; ++j)
      if (used[j]) o << "    const double x" << j << " = sx[" << j << "][lane];\n";
    g.emit_forward(fcone[q], 0, "x", "    ");
    for (int k : part.feat[q]) o << "    sphi[" << fs(k) << "][lane][" << fk(k) << "] = slogf_(v" << d.froots[k] << ");\n";
    o << "    TWSTAMP();\n  }\n";
  }
  o << "  __syncthreads();\n  TSTAMP(0, 3);\n"
    << "  // rows c0 .. c0+31 of each statement are contiguous: K0P/8 uint4 per row for hi and for lo\n"
    << "#pragma unroll\n"
    << "  for (int it = 0; it < (NS * 32 * (K0P / 8) + PG * 32 - 1) / (PG * 32); ++it) {\n"
    << "    const int e0 = tid + it * PG * 32;\n"
    << "    if (e0 >= NS * 32 * (K0P / 8)) break;\n"
    << "    const int st = e0 / (32 * (K0P / 8)), e = e0 % (32 * (K0P / 8));\n"
    << "    const int r = e / (K0P / 8), q8 = e % (K0P / 8);\n"
    << "    if (c0 + r >= n) continue;\n"
    << "    const size_t row = (size_t)st * n + c0 + r;\n"
    << "    u32 h[4], l[4];\n"
    << "#pragma unroll\n"
    << "    for (int u = 0; u < 4; ++u) {\n"
    << "      const float f0 = sphi[st][r][q8 * 8 + 2 * u], f1 = sphi[st][r][q8 * 8 + 2 * u + 1];\n"
    << "      const u16 h0 = f2h(f0), h1 = f2h(f1);\n"
    << "      h[u] = (u32)h0 | ((u32)h1 << 16);\n"
    << "      l[u] = (u32)f2h(f0 - h2f(h0)) | ((u32)f2h(f1 - h2f(h1)) << 16);\n"
    << "    }\n"
    << "    reinterpret_cast<uint4*>(phi_hi + row * K0P)[q8] = make_uint4(h[0], h[1], h[2], h[3]);\n"
    << "    reinterpret_cast<uint4*>(phi_lo + row * K0P)[q8] = make_uint4(l[0], l[1], l[2], l[3]);\n"
    << "  }\n  TSTAMP(0, 4);\n}\n"
    << "#if !defined(FELIX_PART) || FELIX_PART == 1\n"
    << "extern \"C\" __global__ void __launch_bounds__(PG * 32 * NREP) felix_fwd(const float* __restrict__ yv, int n, int ldy, u16* __restrict__ phi_hi, u16* __restrict__ phi_lo, int* step_ctr) {\n"
    << "  fwd_body<0>(const_cast<float*>(yv), n, ldy, phi_hi, phi_lo, step_ctr, nullptr, nullptr, nullptr, nullptr, nullptr, 0, 0, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f);\n}\n#endif\n"
    << "#if !defined(FELIX_PART) || FELIX_PART == 2\n"
    << "extern \"C\" __global__ void __launch_bounds__(PG * 32 * NREP) felix_fwd_adam(float* yv, int n, int ldy, u16* __restrict__ phi_hi, u16* __restrict__ phi_lo, int* step_ctr,\n"
    << "    float* mv, float* vv, const float* __restrict__ part, const double* __restrict__ pen, const float* __restrict__ c_part,\n"
    << "    int n_head_tiles, int ld_c, float head_b, float lam, float lr, float b1, float b2, float eps) {\n"
    << "  fwd_body<1>(yv, n, ldy, phi_hi, phi_lo, step_ctr, mv, vv, part, pen, c_part, n_head_tiles, ld_c, head_b, lam, lr, b1, b2, eps);\n}\n#endif\n\n";

  // ---------------------------------------------------------------- felix_rev (template on mode)
  // smem: partial adjoints of x  spart[PG][NV][32], user-root penalties per group spen[PG][32],
  // auto-root penalties spa[NRA][32], y staged sy[NV][32].
  o << "template <int EVAL>\n__device__ __forceinline__ void rev_body(float* __restrict__ yv, const float* __restrict__ yin, int n, int ldy,\n"
    << "    const float* __restrict__ dphi, int ld_dphi, const float* __restrict__ c_part, int n_head_tiles, int ld_c, float head_b, float lam,\n"
    << "    float* __restrict__ mv, float* __restrict__ vv, const int* step_ctr, float lr, float b1, float b2, float eps,\n"
    << "    float* __restrict__ o_phi, float* __restrict__ o_g, float* __restrict__ o_cost, float* __restrict__ o_loss, float* __restrict__ o_grad,\n"
    << "    double* __restrict__ o_F) {\n"
    << "  extern __shared__ double smem[];\n"
    << "  const int rep = threadIdx.x / (PG * 32), tid = threadIdx.x % (PG * 32);\n"
    << "  constexpr int REPW = ((PG * NV * 32 + PG * 32 + (NRA > 0 ? NRA : 1) * 32) * 8 + NV * 32 * 4 + 15) / 16 * 2;   // doubles per replica\n"
    << "  double* spart = smem + rep * REPW;                     // [PG][NV][32]\n"
    << "  double* spen = spart + PG * NV * 32;                   // [PG][32]\n"
    << "  double* spa = spen + PG * 32;                          // [NRA][32]\n"
    << "  float* sy = reinterpret_cast<float*>(spa + (NRA > 0 ? NRA : 1) * 32);   // [NV][32]\n"
    << "  const int lane = threadIdx.x & 31, wq = tid >> 5;\n"
    << "  const int c0 = (blockIdx.x * NREP + rep) * 32, c = c0 + lane;\n"
    << "  const int cw = c;\n"
    << "  const bool live = c < n;\n"
    << "  const int cc = live ? c : n - 1;\n"
    << "  const bool livew = cw < n;\n"
    << "  const int ccw = livew ? cw : n - 1;\n"
    << "  asm volatile(\"griddepcontrol.launch_dependents;\" ::: \"memory\");\n"
    << "  if (!EVAL) TSTAMP(1, 4);\n"
    << "  asm volatile(\"griddepcontrol.wait;\" ::: \"memory\");\n"
    << "  if (!EVAL) TSTAMP(1, 5);\n"
    << "  const double dlam = (double)lam;\n"
    // everything the epilogue needs from memory is requested now, so its latency overlaps the DAG
    << "  __shared__ double sx_all[NREP][NV * 32];\n"
    << "  double* sx = sx_all[rep];\n"
    << "  for (int e = tid; e < NV * 32; e += PG * 32) { const int j = e >> 5, l = e & 31; const int cl = c0 + l; const float yy = yin[(size_t)j * ldy + (cl < n ? cl : n - 1)]; sy[e] = yy; sx[e] = exp((double)yy); }\n"
    << "  __syncthreads();\n"
    << "  constexpr int NJ = (NV + PG - 1) / PG;   // vars handled by this thread: j = wq + PG * jj\n"
    // Adam state and the head partials go to shared memory with cp.async (no registers held across the
    // DAG, latency hidden behind it); consumed after the cone groups finish
    << "  constexpr int HTMAX = 32;\n"
    << "  __shared__ float smv_all[NREP][2 * NV * 32];\n"
    << "  __shared__ float scp_all[NREP][HTMAX * 32];\n"
    << "  float* smv = smv_all[rep];\n"
    << "  float* scp = scp_all[rep];\n"
    << "  const int nht_all = NS * n_head_tiles;\n"
    << "  const bool cp_smem = nht_all <= HTMAX;\n"
    << "  if (!EVAL) for (int e = tid; e < 2 * NV * 32; e += PG * 32) { const int h = e / (NV * 32), j = (e >> 5) % NV, l = e & 31; const int cl = c0 + l < n ? c0 + l : n - 1; cp_async4(&smv[e], (h ? vv : mv) + (size_t)j * n + cl); }\n"
    << "  if (cp_smem) for (int e = tid; e < nht_all * 32; e += PG * 32) { const int i = e >> 5, l = e & 31; const int cl = c0 + l < n ? c0 + l : n - 1; cp_async4(&scp[e], c_part + (size_t)(i % n_head_tiles) * ld_c + (size_t)(i / n_head_tiles) * n + cl); }\n"
    << "  cp_async_commit();\n"
    << "  const int tstep = EVAL ? 1 : *step_ctr;\n";
  // Per cone: with EVAL, the FP64 search forward (mode 0) for the phi / F / g outputs; then, in both
  // kernels, the FP32 forward recompute + FP32 reverse sweep of the search (DESIGN.md "Precision of the
  // expression kernels"), penalties and partial adjoints to shared memory.
  for (int q = 0; q < P; ++q) {
    o << "  if (wq == " << q << ") {\n";
    const auto used = vars_in(rcone[q]);
    o << "    if constexpr (EVAL) {\n";
    if (q == 0) {
      o << "    if ((o_phi || o_F) && livew) {\n";
      for (int k = 0; k < K; ++k)
        if (!g.depvar[d.froots[k]]) {
          o << "      {\n";
          g.emit_forward(g.cone({d.froots[k]}), 0, "x", "        ");
          o << "        if (o_phi) o_phi[(size_t)" << k << " * n + cw] = slogf_(v" << d.froots[k] << ");\n"
            << "        if (o_F) o_F[(size_t)" << k << " * n + cw] = v" << d.froots[k] << ";\n      }\n";
        }
      o << "    }\n";
    }
    for (int j = 0; j < M; ++j)
      if (used[j]) o << "    const double x" << j << " = sx[" << j << " * 32 + lane];\n";
    g.emit_forward(rcone[q], 0, "x", "    ");
    for (int r : part.cons[q]) o << "    if (o_g && livew) o_g[(size_t)" << r << " * n + cw] = (float)v" << d.croots[r] << ";\n";
    o << "    if (o_phi && livew) {\n";
    for (int k : part.feat[q]) o << "      o_phi[(size_t)" << k << " * n + cw] = slogf_(v" << d.froots[k] << ");\n";
    o << "    }\n";
    o << "    if (o_F && livew) {\n";
    for (int k : part.feat[q]) o << "      o_F[(size_t)" << k << " * n + cw] = v" << d.froots[k] << ";\n";
    o << "    }\n";
    o << "    }\n    {\n";
    for (int j = 0; j < M; ++j)
      if (used[j]) o << "    const float x" << j << " = expf(sy[" << j << " * 32 + lane]);\n";
    g.emit_forward(rcone[q], 3, "x", "    ");
    // user-root penalties of this group
    o << "    float pen = 0.f;\n";
    for (int r : part.cons[q]) o << "    const float p" << r << " = fmaxf(v" << d.croots[r] << ", 0.f); pen += p" << r << " * p" << r << ";\n";
    o << "    spen[" << q << " * 32 + lane] = (double)pen;\n";
    const auto need = g.rev_live(rcone[q], rroots_g[q]);
    g.emit_adj_decls(need, "    ", true);
    for (int j = 0; j < M; ++j) o << "    float gx" << j << " = 0.f;\n";
    for (int k : part.feat[q]) {
      const int r = d.froots[k];
      o << "    " << g.adj(r) << " += " << dphi_at("(size_t)" + std::to_string(fk(k)) + " * ld_dphi + (size_t)" +
                                                  std::to_string(fs(k)) + " * n + ccw") << " * slogpf_(v" << r << ");\n";
    }
    for (int r : part.cons[q]) {
      const int nd = d.croots[r];
      if (g.depvar[nd]) o << "    " << g.adj(nd) << " += 2.f * lam * p" << r << ";\n";
    }
    g.emit_reverse_body(need, "    ", true);
    for (int j = 0; j < M; ++j) o << "    spart[(" << q << " * NV + " << j << ") * 32 + lane] = (double)gx" << j << ";\n";
    o << "    }\n  }\n";
  }
  // automatic roots (warp 0) from the staged y
  o << "  cp_async_wait_all();\n  __syncthreads();\n  if (!EVAL) TSTAMP(1, 6);\n"
    << "  if (wq == 0) {\n";
  for (int j = 0; j < M; ++j) o << "    const double y" << j << " = (double)sy[" << j << " * 32 + lane];\n";
  for (size_t q = 0; q < autos.size(); ++q) {
    o << "    { const double gr = " << autos[q].val << "; spa[" << q << " * 32 + lane] = fmax(gr, 0.0);\n"
      << "      if (EVAL && o_g && live) o_g[(size_t)" << Ru + (int)q << " * n + c] = (float)gr; }\n";
  }
  o << "  }\n  __syncthreads();\n";
  // cost + loss (warp 0); the loss is parked in spen[PG-1 .. ] row 0 after the sum
  o << "  __shared__ float sloss_all[NREP][32];\n  float* sloss = sloss_all[rep];\n"
    << "  if (wq == 0) {\n"
    << "    float cst = head_b * NS;   // segment sum over statements: every statement's MLP adds its head bias\n"
    << "    if (cp_smem) for (int i = 0; i < nht_all; ++i) cst += scp[i * 32 + lane];\n"
    << "    else for (int s = 0; s < NS; ++s) for (int t = 0; t < n_head_tiles; ++t) cst += c_part[(size_t)t * ld_c + (size_t)s * n + cc];\n"
    << "    double pen = 0.0;\n"
    << "    for (int q = 0; q < PG; ++q) pen += spen[q * 32 + lane];\n"
    << "    for (int r = 0; r < NRA; ++r) { const double p = spa[r * 32 + lane]; pen += p * p; }\n"
    << "    const float loss = (float)(-(double)cst + dlam * pen);\n"
    << "    sloss[lane] = loss;\n"
    << "    if (live) {\n      if (o_loss) o_loss[c] = loss;\n      if (EVAL && o_cost) o_cost[c] = cst;\n    }\n  }\n";
  // gradient per (var, candidate): thread (wq, lane) handles vars j = wq, wq + PG, ...
  o << "  __shared__ float sgrad_all[NREP][NV][32];\n  float (&sgrad)[NV][32] = sgrad_all[rep];\n"
    << "#pragma unroll\n"
    << "  for (int jj = 0; jj < NJ; ++jj) {\n"
    << "    const int j = wq + PG * jj;\n"
    << "    if (j >= NV) break;\n"
    << "    double gx = 0.0;\n"
    << "    for (int q = 0; q < PG; ++q) gx += spart[(q * NV + j) * 32 + lane];\n"
    << "    double gd = sx[j * 32 + lane] * gx;\n"
    << "    switch (j) {\n";
  for (int j = 0; j < M; ++j) {
    std::string terms;
    for (size_t q = 0; q < autos.size(); ++q)
      for (auto& tv : autos[q].terms)
        if (tv.first == j) terms += std::string(tv.second > 0 ? " + " : " - ") + "spa[" + std::to_string(q) + " * 32 + lane]";
    if (!terms.empty()) o << "      case " << j << ": gd += 2.0 * dlam * (0.0" << terms << "); break;\n";
  }
  o << "      default: break;\n    }\n"
    << "    const float gy = (float)gd;\n"
    << "    sgrad[j][lane] = gy;\n"
    << "    if (EVAL) { if (o_grad && live) o_grad[(size_t)j * n + c] = gy; }\n"
    << "  }\n";
  // R-NaN: the candidate is updated only if its loss and every gradient component are finite
  o << "  if (!EVAL) {\n"
    << "    __syncthreads();\n"
    << "    bool ok = isfinite(sloss[lane]);\n"
    << "    for (int j = 0; j < NV; ++j) ok = ok && isfinite(sgrad[j][lane]);\n"
    << "    if (ok && live) {\n"
    << "      const float bc1 = 1.f - powf(b1, (float)tstep), bc2 = 1.f - powf(b2, (float)tstep);\n"
    << "      const float step = lr / bc1, rb = 1.f / sqrtf(bc2);\n"
    << "#pragma unroll\n"
    << "      for (int jj = 0; jj < NJ; ++jj) {\n"
    << "        const int j = wq + PG * jj;\n"
    << "        if (j >= NV) break;\n"
    << "        const float gy = sgrad[j][lane];\n"
    << "        const size_t o_ = (size_t)j * n + c;\n"
    << "        float m = smv[j * 32 + lane], v = smv[(NV + j) * 32 + lane];\n"
    << "        m = b1 * m + (1.f - b1) * gy; v = b2 * v + (1.f - b2) * gy * gy;\n"
    << "        mv[o_] = m; vv[o_] = v; yv[(size_t)j * ldy + c] = sy[j * 32 + lane] - step * m / (sqrtf(v) * rb + eps);\n"
    << "      }\n"
    << "    }\n"
    << "    TSTAMP(1, 7);\n"
    << "  }\n}\n\n";
  o << "#if !defined(FELIX_PART) || FELIX_PART == 3\n" "extern \"C\" __global__ void __launch_bounds__(PG * 32 * NREP) felix_rev_adam(float* yv, int n, int ldy, const float* dphi, int ld_dphi, const float* c_part, int n_head_tiles, int ld_c, float head_b, float lam,\n"
    << "    float* mv, float* vv, const int* step_ctr, float lr, float b1, float b2, float eps, float* o_loss) {\n"
    << "  rev_body<0>(yv, yv, n, ldy, dphi, ld_dphi, c_part, n_head_tiles, ld_c, head_b, lam, mv, vv, step_ctr, lr, b1, b2, eps, nullptr, nullptr, nullptr, o_loss, nullptr, nullptr);\n}\n#endif\n";
  o << "#if !defined(FELIX_PART) || FELIX_PART == 4\n" "extern \"C\" __global__ void __launch_bounds__(PG * 32 * NREP) felix_rev_eval(const float* yv, int n, int ldy, const float* dphi, int ld_dphi, const float* c_part, int n_head_tiles, int ld_c, float head_b, float lam,\n"
    << "    float* o_phi, float* o_g, float* o_cost, float* o_loss, float* o_grad, double* o_F) {\n"
    << "  rev_body<1>(nullptr, yv, n, ldy, dphi, ld_dphi, c_part, n_head_tiles, ld_c, head_b, lam, nullptr, nullptr, nullptr, 0.f, 0.f, 0.f, 0.f, o_phi, o_g, o_cost, o_loss, o_grad, o_F);\n}\n#endif\n\n";

  // ---------------------------------------------------------------- split-cone search kernels
  // felix_rev_sc runs ONE cone per CTA (block-uniform q = blockIdx.x % PG) for W x 32 candidates, so the
  // warps of an SM share one cone's straight-line code and instruction fetches (felix_rev_adam puts P
  // different cones in one CTA and is instruction-fetch bound: 42 % of its stall samples are
  // no_instructions).  Cone q's CTA writes its partial adjoints part[q][j][c] = x_j dL/dx_j = this cone's dL/dy_j (x_j folded in) and its user-root
  // penalty pen[q][c]; the cross-cone sums and Adam happen after the kernel boundary: in the next step's
  // forward (felix_fwd_adam, whose CTAs own whole candidates) and, after the last step, in felix_adam_sc.
  // Step counter: starts at 1, felix_rev_sc adds 1 (block 0, after griddepcontrol.wait; no CTA of the
  // reverse kernel reads it), so the forward and the MLP chain of step t see t and Adam step t - 1 is due.
  // Measured and dropped: Adam by the last of the P cone CTAs to arrive (+8 us at C2: a serial tail at
  // 255 registers), and a split-cone forward (its 2-byte feature-column stores: 1.7x slower at C2).
  // The whole kernel is FP32 (forward recompute, seeds, reverse sweep): its outputs are gradients, whose
  // tolerance is 1e-3; half the registers and a third
  // of the instructions of the FP64 form, so the straight-line cone code streams through the SM's
  // instruction fetch faster.
  o << "#if !defined(FELIX_PART) || FELIX_PART == 5\n" "extern \"C\" __global__ void __launch_bounds__(256) felix_rev_sc(const float* __restrict__ yv, int n, int ldy, const float* __restrict__ dphi, int ld_dphi,\n"
    << "    float lam, float* __restrict__ part, double* __restrict__ pen, int* step_ctr) {\n"
    << "  const int cq_ = blockIdx.x % PG;\n"
    << "  const int c = ((blockIdx.x / PG) * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 32 + (threadIdx.x & 31);\n"
    << "  const bool live = c < n;\n  const int ccw = live ? c : n - 1;\n"
    << "  asm volatile(\"griddepcontrol.launch_dependents;\" ::: \"memory\");\n"
    << "  TSTAMP(1, 0);\n"
    << "  asm volatile(\"griddepcontrol.wait;\" ::: \"memory\");\n"
    << "  TSTAMP(1, 1);\n"
    << "  if (blockIdx.x == 0 && threadIdx.x == 0) *step_ctr += 1;\n";
  for (int q = 0; q < P; ++q) {
    o << "  if (cq_ == " << q << ") {\n";
    const auto used = vars_in(rcone[q]);
    for (int j = 0; j < M; ++j)
      if (used[j]) o << "    const float x" << j << " = expf(yv[(size_t)" << j << " * ldy + ccw]);\n";
    g.emit_forward(rcone[q], 3, "x", "    ");
    o << "    float pq = 0.f;\n";
    for (int r : part.cons[q]) o << "    const float pr" << r << " = fmaxf(v" << d.croots[r] << ", 0.f); pq += pr" << r << " * pr" << r << ";\n";
    const auto need = g.rev_live(rcone[q], rroots_g[q]);
    g.emit_adj_decls(need, "    ", true);
    for (int j = 0; j < M; ++j) o << "    float gx" << j << " = 0.f;\n";
    for (int k : part.feat[q]) {
      const int r = d.froots[k];
      o << "    " << g.adj(r) << " += " << dphi_at("(size_t)" + std::to_string(fk(k)) + " * ld_dphi + (size_t)" +
                                                  std::to_string(fs(k)) + " * n + ccw") << " * slogpf_(v" << r << ");\n";
    }
    for (int r : part.cons[q]) {
      const int nd = d.croots[r];
      if (g.depvar[nd]) o << "    " << g.adj(nd) << " += 2.f * lam * pr" << r << ";\n";
    }
    g.emit_reverse_body(need, "    ", true);
    o << "    TSTAMP(1, 2);\n";
    // partial dL/dy_j = x_j * dL/dx_j of this cone (x_j is at hand here; the Adam prologue needs no exp)
    o << "    if (live) {\n      pen[(size_t)" << q << " * n + c] = (double)pq;\n";
    for (int j = 0; j < M; ++j)
      o << "      part[((size_t)" << q << " * NV + " << j << ") * n + c] = " << (used[j] ? "x" + std::to_string(j) + " * gx" + std::to_string(j) : std::string("0.f")) << ";\n";
    o << "    }\n    TSTAMP(1, 3);\n  }\n";
  }
  o << "}\n#endif\n\n";
  // felix_adam_sc: the last Adam step (thread per candidate, in place) + the final loss
  o << "#if !defined(FELIX_PART) || FELIX_PART == 6\n" "extern \"C\" __global__ void __launch_bounds__(128) felix_adam_sc(float* yv, int n, int ldy, float* mv, float* vv,\n"
    << "    const float* __restrict__ part, const double* __restrict__ pen, const float* __restrict__ c_part, int n_head_tiles, int ld_c,\n"
    << "    float head_b, float lam, float lr, float b1, float b2, float eps, const int* step_ctr, float* o_loss, float* o_grad) {\n"
    << "  const int c = blockIdx.x * blockDim.x + threadIdx.x;\n  if (c >= n) return;\n"
    << "  const int s_ = *step_ctr - 1;\n  if (s_ <= 0) return;\n"
    << "  const double dlam = (double)lam;\n"
    << "  float syv[NV], ml[NV], vl[NV], gxa[NV];\n"
    << "#pragma unroll\n  for (int j = 0; j < NV; ++j) {\n"
    << "    syv[j] = yv[(size_t)j * ldy + c]; ml[j] = mv[(size_t)j * n + c]; vl[j] = vv[(size_t)j * n + c];\n"
    << "    float a = 0.f;\n#pragma unroll\n    for (int q = 0; q < PG; ++q) a += part[((size_t)q * NV + j) * n + c];\n"
    << "    gxa[j] = a;\n  }\n"
    << "  double pen_ = 0.0;\n#pragma unroll\n  for (int q = 0; q < PG; ++q) pen_ += pen[(size_t)q * n + c];\n"
    << "  float cst = head_b * NS;\n"
    << "  for (int i = 0; i < NS * n_head_tiles; ++i) cst += c_part[(size_t)(i % n_head_tiles) * ld_c + (size_t)(i / n_head_tiles) * n + c];\n";
  emit_autos("  ", "syv");
  o << "  const float loss = (float)(-(double)cst + dlam * pen_);\n"
    << "  if (o_loss) o_loss[c] = loss;\n"
    << "  bool ok = isfinite(loss);\n  float gy[NV];\n"
    << "#pragma unroll\n  for (int j = 0; j < NV; ++j) {\n"
    << "    double gd = (double)gxa[j];\n";
  emit_auto_grad_switch("    ");
  o << "    gy[j] = (float)gd;\n    ok = ok && isfinite(gy[j]);\n  }\n"
    << "  if (o_grad) {   // test hook (felix_eval_ex search_path): dL/dy as the search's Adam step sees it, no update\n"
    << "#pragma unroll\n    for (int j = 0; j < NV; ++j) o_grad[(size_t)j * n + c] = gy[j];\n    return;\n  }\n"
    << "  if (!ok) return;\n"
    << "  const float bc1 = 1.f - powf(b1, (float)s_), bc2 = 1.f - powf(b2, (float)s_);\n"
    << "  const float step = lr / bc1, rb = 1.f / sqrtf(bc2);\n"
    << "#pragma unroll\n  for (int j = 0; j < NV; ++j) {\n"
    << "    float m = ml[j], v = vl[j];\n"
    << "    m = b1 * m + (1.f - b1) * gy[j]; v = b2 * v + (1.f - b2) * gy[j] * gy[j];\n"
    << "    mv[(size_t)j * n + c] = m; vv[(size_t)j * n + c] = v; yv[(size_t)j * ldy + c] = syv[j] - step * m / (sqrtf(v) * rb + eps);\n"
    << "  }\n}\n#endif\n\n";

  // ---------------------------------------------------------------- felix_hard (fp64 IEEE, integer points)
  std::vector<bool> all(g.n, true);
  o << "#if !defined(FELIX_PART) || FELIX_PART == 7\n" "extern \"C\" __global__ void __launch_bounds__(128) felix_hard(const int* __restrict__ sched, int n, double* __restrict__ phi64, unsigned char* __restrict__ valid) {\n"
    << "  const int i = blockIdx.x * blockDim.x + threadIdx.x;\n  if (i >= n) return;\n";
  for (int j = 0; j < M; ++j) o << "  const double h" << j << " = (double)sched[(size_t)i * NV + " << j << "];\n";
  g.emit_forward(all, 2, "h");
  o << "  bool ok = true;\n";
  for (int k = 0; k < K; ++k)
    o << "  ok = ok && isfinite(v" << d.froots[k] << "); phi64[(size_t)" << k << " * n + i] = slogd_(v" << d.froots[k] << ");\n";
  for (int r = 0; r < Ru; ++r) o << "  ok = ok && isfinite(v" << d.croots[r] << ") && (v" << d.croots[r] << " <= 1e-9);\n";
  o << "  valid[i] = ok ? 1 : 0;\n}\n#endif\n\n";

  // ---------------------------------------------------------------- felix_init (rejection sampler)
  std::vector<int> parent(M);
  std::iota(parent.begin(), parent.end(), 0);
  std::function<int(int)> find = [&](int j) { while (parent[j] != j) { parent[j] = parent[parent[j]]; j = parent[j]; } return j; };
  for (auto& sv : d.split_vars) for (size_t k = 1; k < sv.size(); ++k) parent[find(sv[k])] = find(sv[0]);
  std::vector<std::vector<int>> comps;
  {
    std::vector<int> root_of(M, -1);
    for (int j = 0; j < M; ++j) {
      if (d.vars[j].kind != FELIX_VAR_SPLIT) continue;
      const int r = find(j);
      if (root_of[r] < 0) { root_of[r] = (int)comps.size(); comps.push_back({}); }
      comps[root_of[r]].push_back(j);
    }
  }
  // one warp per candidate: lane L evaluates outer attempt a2 = base + L (a pure function of a2), the
  // first accepted attempt in attempt order wins (ballot) and its y is broadcast: the same starting point
  // as the serial rejection loop of the spec, with the serial chain of attempts replaced by 32 in flight
  o << "#if !defined(FELIX_PART) || FELIX_PART == 8\n" "extern \"C\" __global__ void __launch_bounds__(128) felix_init(u64 seed, int n, long long index_base, float* __restrict__ yout) {\n"
    << "  const int lane = threadIdx.x & 31;\n"
    << "  const int i = (int)(((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5);\n  if (i >= n) return;\n"
    << "  const u64 cand = (u64)(index_base + i);\n";
  for (int j = 0; j < M; ++j) o << "  double y" << j << " = 0.0;\n";
  o << "  int win = -1;\n  for (int base = 0; base < 64 && win < 0; base += 32) {\n    const int a2 = base + lane;\n";
  for (const auto& comp : comps) {
    o << "    {\n      bool acc = false;\n";
    for (int j : comp) o << "      double c" << j << " = 0.0;\n";
    o << "      for (int a1 = 0; a1 < 64 && !acc; ++a1) {\n        const u64 att = (u64)(a2 * 64 + a1);\n";
    for (int j : comp) {
      double ub = 1e300;
      for (size_t s = 0; s < d.split_vars.size(); ++s)
        for (int v : d.split_vars[s]) if (v == j) ub = std::min(ub, (double)d.split_extent[s]);
      o << "        const double t" << j << " = __dmul_rn(cuni(seed, cand, att, " << j << "ull), " << lit(std::log(ub)) << ");\n";
    }
    o << "        bool ok = true;\n";
    for (size_t s = 0; s < d.split_vars.size(); ++s) {
      bool mine = false;
      for (int v : d.split_vars[s]) for (int j : comp) if (v == j) mine = true;
      if (!mine) continue;
      o << "        { double tot = 0.0;";
      for (int v : d.split_vars[s]) o << " tot = __dadd_rn(tot, t" << v << ");";
      o << " ok = ok && (__dsub_rn(tot, " << lit(std::log((double)d.split_extent[s])) << ") <= 0.0); }\n";
    }
    o << "        if (ok) { acc = true;";
    for (int j : comp) o << " c" << j << " = t" << j << ";";
    o << " }\n      }\n";
    for (int j : comp) o << "      y" << j << " = c" << j << ";\n";
    o << "    }\n";
  }
  for (int j = 0; j < M; ++j) {
    if (d.vars[j].kind != FELIX_VAR_INT) continue;
    const double llo = std::log((double)d.vars[j].lo), lhi = std::log((double)d.vars[j].hi);
    o << "    y" << j << " = __dadd_rn(" << lit(llo) << ", __dmul_rn(cuni(seed, cand, (u64)(a2 * 64), " << j << "ull), "
      << lit(lhi - llo) << "));\n";
  }
  o << "    bool ok = true;\n    {\n";
  for (int j = 0; j < M; ++j) o << "      const double x" << j << " = exp(y" << j << ");\n";
  std::vector<int> cr(d.croots.begin(), d.croots.end());
  g.emit_forward(g.cone(cr), 1, "x", "      ");
  for (int r = 0; r < Ru; ++r) o << "      ok = ok && (v" << d.croots[r] << " <= 0.0);\n";
  o << "    }\n"
    << "    const unsigned acc_mask = __ballot_sync(0xffffffffu, ok);\n"
    << "    if (acc_mask) {\n      const int src = __ffs(acc_mask) - 1;\n      win = base + src;\n";
  for (int j = 0; j < M; ++j) o << "      y" << j << " = __shfl_sync(0xffffffffu, y" << j << ", src);\n";
  o << "    }\n  }\n  if (win < 0) {\n";
  for (int j = 0; j < M; ++j)
    o << "    y" << j << " = " << (d.vars[j].kind == FELIX_VAR_INT ? lit(std::log((double)d.vars[j].lo)) : "0.0") << ";\n";
  o << "  }\n";
  for (int j = 0; j < M; ++j) o << "  if (lane == " << (j % 32) << ") yout[(size_t)" << j << " * n + i] = (float)y" << j << ";\n";
  o << "}\n#endif\n\n";

  if (info) {
    info->flops_fwd = flops_fwd;
    info->flops_rev = flops_rev;
    info->rev_smem_bytes = NREPv * (((P * M * 32 + P * 32 + std::max(Ra, 1) * 32) * 8 + M * 32 * 4 + 15) / 16 * 16);
  }
  return o.str();
}

}  // namespace felix
