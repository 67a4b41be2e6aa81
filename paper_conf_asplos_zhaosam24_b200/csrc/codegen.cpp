// codegen.cpp — per-space straight-line CUDA for the feature-expression DAG, compiled with NVRTC.
//
// Felix's expression rewriter (Rust + egg, L1068-1071) turns feature formulas into
// smooth differentiable expressions, takes their logarithm and substitutes x = e^y.  Here the same
// rewrite is *emitted as code*: one candidate per thread, every DAG node a named register value,
// the reverse sweep (Alg. 1 line 18) as straight-line adjoint statements, fused with the
// loss / penalty seeds (Eq. 4) and the Adam update (L889-892).  Generated kernels:
//   felix_fwd        smooth fp32 forward -> phi = slog(F) as fp16 hi/lo rows (MMA A operand)
//   felix_rev_adam   recompute forward, seeds, reverse sweep, dL/dy, Adam (fp32)
//   felix_rev_eval   same, writing phi / g / cost / loss / grad instead of updating y
//   felix_hard       hard semantics in fp64 at integer points -> slog features (fp64) + validity
//   felix_init       rejection sampler (fp64 decisions, counter-based RNG)
#include <cmath>
#include <cstdio>
#include <functional>
#include <sstream>
#include <string>
#include <vector>
#include "felix_internal.h"

namespace felix {

namespace {

std::string lit(double v, bool dbl) {
  if (std::isinf(v)) return v > 0 ? (dbl ? "(1.0/0.0)" : "(1.0f/0.0f)") : (dbl ? "(-1.0/0.0)" : "(-1.0f/0.0f)");
  char buf[64];
  if (dbl) snprintf(buf, sizeof buf, "%.17g", v);
  else snprintf(buf, sizeof buf, "%.9gf", (double)(float)v);
  std::string s(buf);
  if (dbl && s.find_first_of(".eEn") == std::string::npos) s += ".0";
  if (!dbl && s.find_first_of(".eEn") == std::string::npos) s.insert(s.size() - 1, ".0");
  return s;
}

const char* kPrelude = R"CUDA(
typedef unsigned long long u64;
typedef unsigned int u32;
typedef unsigned short u16;
#define LN2F 0.693147180559945309f
__device__ __forceinline__ u16 f2h(float f) { u16 h; asm("cvt.rn.f16.f32 %0, %1;" : "=h"(h) : "f"(f)); return h; }
__device__ __forceinline__ float h2f(u16 h) { float f; asm("cvt.f32.f16 %0, %1;" : "=f"(f) : "h"(h)); return f; }
// smoothing kernel phi(t) = 1/2 (1+t^2)^(-3/2) (reading O3): S = step * phi, R = relu * phi
__device__ __forceinline__ float sm_hyp(float t) { float a = fabsf(t); if (a > 1.f) { float r = 1.f / a; return a * sqrtf(1.f + r * r); } return sqrtf(1.f + t * t); }
__device__ __forceinline__ double sm_hyp(double t) { double a = fabs(t); if (a > 1.0) { double r = 1.0 / a; return a * sqrt(1.0 + r * r); } return sqrt(1.0 + t * t); }
__device__ __forceinline__ float sm_S(float t) { float h = sm_hyp(t), a = fabsf(t); float tail = 1.f / (2.f * h * (h + a)); return t >= 0.f ? 1.f - tail : tail; }
__device__ __forceinline__ double sm_S(double t) { double h = sm_hyp(t), a = fabs(t); double tail = 1.0 / (2.0 * h * (h + a)); return t >= 0.0 ? 1.0 - tail : tail; }
__device__ __forceinline__ float sm_dS(float t) { float h = sm_hyp(t); return 0.5f / (h * h * h); }
__device__ __forceinline__ double sm_dS(double t) { double h = sm_hyp(t); return 0.5 / (h * h * h); }
// R(t) - relu(t) = 1/(2(sqrt(1+t^2) + |t|)); min / max without the cancellation of a - (a - b)
__device__ __forceinline__ float sm_gap(float t) { float h = sm_hyp(t); return 1.f / (2.f * (h + fabsf(t))); }
__device__ __forceinline__ double sm_gap(double t) { double h = sm_hyp(t); return 1.0 / (2.0 * (h + fabs(t))); }
__device__ __forceinline__ float sm_min(float a, float b) { const float t = a - b; return (t >= 0.f ? b : a) - sm_gap(t); }
__device__ __forceinline__ double sm_min(double a, double b) { const double t = a - b; return (t >= 0.0 ? b : a) - sm_gap(t); }
__device__ __forceinline__ float sm_max(float a, float b) { const float t = a - b; return (t >= 0.f ? a : b) + sm_gap(t); }
__device__ __forceinline__ double sm_max(double a, double b) { const double t = a - b; return (t >= 0.0 ? a : b) + sm_gap(t); }
__device__ __forceinline__ float p_pow(float a, float e) { return powf(a, e); }
__device__ __forceinline__ double p_pow(double a, double e) { return pow(a, e); }
__device__ __forceinline__ float p_exp(float a) { return expf(a); }
__device__ __forceinline__ double p_exp(double a) { return exp(a); }
__device__ __forceinline__ float p_log(float a) { return logf(a); }
__device__ __forceinline__ double p_log(double a) { return log(a); }
__device__ __forceinline__ float p_sqrt(float a) { return sqrtf(a); }
__device__ __forceinline__ double p_sqrt(double a) { return sqrt(a); }
// slog(F) = sign(F) log2(1 + |F|)  (reading O4)
__device__ __forceinline__ float slogf_(float f) { float l = log2f(1.f + fabsf(f)); return f < 0.f ? -l : l; }
__device__ __forceinline__ float slogpf_(float f) { return 1.f / ((1.f + fabsf(f)) * LN2F); }
__device__ __forceinline__ double slogd_(double f) { double l = log2(1.0 + fabs(f)); return f < 0.0 ? -l : (f > 0.0 ? l : 0.0); }
__device__ __forceinline__ double slogpd_(double f) { return 1.0 / ((1.0 + fabs(f)) * 0.69314718055994530942); }
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

struct Gen {
  const SpaceDesc& d;
  int n;
  std::vector<bool> depvar;     // node depends on a variable
  std::vector<bool> needed_rev; // node receives an adjoint
  std::ostringstream o;
  int64_t flops = 0;

  explicit Gen(const SpaceDesc& dd) : d(dd), n((int)dd.nodes.size()), depvar(n, false), needed_rev(n, false) {
    for (int i = 0; i < n; ++i) {
      const felix_node& nd = d.nodes[i];
      if (nd.op == FELIX_OP_VAR) { depvar[i] = true; continue; }
      if (nd.op == FELIX_OP_CONST) continue;
      int ar = arity(nd.op);
      bool dv = false;
      if (ar >= 1) dv |= depvar[nd.a];
      if (ar >= 2) dv |= depvar[nd.b];
      if (ar >= 3) dv |= depvar[nd.c];
      depvar[i] = dv;
    }
    for (int r : d.froots) if (depvar[r]) needed_rev[r] = true;
    for (int r : d.croots) if (depvar[r]) needed_rev[r] = true;
    for (int i = n - 1; i >= 0; --i) {
      if (!needed_rev[i]) continue;
      const felix_node& nd = d.nodes[i];
      int ar = arity(nd.op);
      if (nd.op == FELIX_OP_VAR || nd.op == FELIX_OP_CONST) continue;
      if (ar >= 1 && depvar[nd.a]) needed_rev[nd.a] = true;
      if (ar >= 2 && depvar[nd.b]) needed_rev[nd.b] = true;
      if (ar >= 3 && depvar[nd.c]) needed_rev[nd.c] = true;
    }
  }

  static int arity(int op) {
    switch (op) {
      case FELIX_OP_CONST: case FELIX_OP_VAR: return 0;
      case FELIX_OP_NEG: case FELIX_OP_EXP: case FELIX_OP_LOG: case FELIX_OP_SQRT: case FELIX_OP_NOT: case FELIX_OP_POW: return 1;
      case FELIX_OP_SELECT: return 3;
      default: return 2;
    }
  }

  // forward node values. T = "float"/"double"; hard = exact (integer-point) semantics.
  void emit_forward(bool dbl, bool hard, const char* xname) {
    const char* T = dbl ? "double" : "float";
    const std::string one = dbl ? "1.0" : "1.f";
    const std::string half = dbl ? "0.5" : "0.5f";
    for (int i = 0; i < n; ++i) {
      const felix_node& nd = d.nodes[i];
      std::string A = "v" + std::to_string(nd.a), B = "v" + std::to_string(nd.b), C = "v" + std::to_string(nd.c);
      std::string e;
      switch (nd.op) {
        case FELIX_OP_CONST: e = lit(nd.imm, dbl); break;
        case FELIX_OP_VAR: e = std::string(xname) + std::to_string((int)nd.imm); break;
        case FELIX_OP_ADD: e = A + " + " + B; ++flops; break;
        case FELIX_OP_SUB: e = A + " - " + B; ++flops; break;
        case FELIX_OP_MUL: e = A + " * " + B; ++flops; break;
        case FELIX_OP_DIV: e = A + " / " + B; ++flops; break;
        case FELIX_OP_NEG: e = "-" + A; break;
        case FELIX_OP_POW: e = "p_pow(" + A + ", " + lit(nd.imm, dbl) + ")"; ++flops; break;
        case FELIX_OP_EXP: e = "p_exp(" + A + ")"; ++flops; break;
        case FELIX_OP_LOG: e = "p_log(" + A + ")"; ++flops; break;
        case FELIX_OP_SQRT: e = "p_sqrt(" + A + ")"; ++flops; break;
        case FELIX_OP_MIN: e = hard ? "fmin(" + A + ", " + B + ")" : "sm_min(" + A + ", " + B + ")"; flops += 6; break;
        case FELIX_OP_MAX: e = hard ? "fmax(" + A + ", " + B + ")" : "sm_max(" + A + ", " + B + ")"; flops += 6; break;
        case FELIX_OP_GT: e = hard ? "(" + A + " > " + B + " ? 1.0 : 0.0)" : "sm_S(" + A + " - " + B + ")"; flops += 6; break;
        case FELIX_OP_GE: e = hard ? "(" + A + " >= " + B + " ? 1.0 : 0.0)" : "sm_S(" + A + " - " + B + ")"; flops += 6; break;
        case FELIX_OP_LT: e = hard ? "(" + A + " < " + B + " ? 1.0 : 0.0)" : "sm_S(" + B + " - " + A + ")"; flops += 6; break;
        case FELIX_OP_LE: e = hard ? "(" + A + " <= " + B + " ? 1.0 : 0.0)" : "sm_S(" + B + " - " + A + ")"; flops += 6; break;
        case FELIX_OP_EQ: e = hard ? "(" + A + " == " + B + " ? 1.0 : 0.0)"
                                   : "sm_S((" + A + " - " + B + ") + " + half + ") * sm_S(" + half + " - (" + A + " - " + B + "))"; flops += 12; break;
        case FELIX_OP_NE: e = hard ? "(" + A + " != " + B + " ? 1.0 : 0.0)"
                                   : one + " - sm_S((" + A + " - " + B + ") + " + half + ") * sm_S(" + half + " - (" + A + " - " + B + "))"; flops += 13; break;
        case FELIX_OP_AND: e = A + " * " + B; ++flops; break;
        case FELIX_OP_OR: e = A + " + " + B + " - " + A + " * " + B; flops += 3; break;
        case FELIX_OP_NOT: e = one + " - " + A; ++flops; break;
        case FELIX_OP_SELECT: e = hard ? "(" + A + " != 0.0 ? " + B + " : " + C + ")" : C + " + (" + B + " - " + C + ") * " + A; flops += 3; break;
        case FELIX_OP_FLOORDIV: e = hard ? "floor(" + A + " / " + B + ")" : A + " / " + B; ++flops; break;
        case FELIX_OP_CEILDIV: e = hard ? "ceil(" + A + " / " + B + ")" : A + " / " + B; ++flops; break;
        default: e = "0"; break;
      }
      o << "  const " << T << " v" << i << " = " << e << ";\n";
    }
  }

  // reverse sweep (fp32 smooth). Adjoint of VAR j accumulates into gx<j>.
  void emit_reverse() {
    for (int i = 0; i < n; ++i)
      if (needed_rev[i] && d.nodes[i].op != FELIX_OP_VAR) o << "  double a" << i << " = 0.0;\n";
    for (int j = 0; j < d.n_vars; ++j) o << "  double gx" << j << " = 0.0;\n";
  }
  void emit_reverse_body() {
    auto acc = [&](int tgt, const std::string& expr, bool neg = false) {
      if (!depvar[tgt]) return;
      const felix_node& t = d.nodes[tgt];
      std::string dst = t.op == FELIX_OP_VAR ? "gx" + std::to_string((int)t.imm) : "a" + std::to_string(tgt);
      o << "    " << dst << (neg ? " -= " : " += ") << expr << ";\n";
    };
    for (int i = n - 1; i >= 0; --i) {
      const felix_node& nd = d.nodes[i];
      if (!needed_rev[i] || nd.op == FELIX_OP_VAR || nd.op == FELIX_OP_CONST) continue;
      std::string g = "a" + std::to_string(i);
      std::string A = "v" + std::to_string(nd.a), B = "v" + std::to_string(nd.b), C = "v" + std::to_string(nd.c);
      std::string V = "v" + std::to_string(i);
      o << "  {\n";
      switch (nd.op) {
        case FELIX_OP_ADD: acc(nd.a, g); acc(nd.b, g); break;
        case FELIX_OP_SUB: acc(nd.a, g); acc(nd.b, g, true); break;
        case FELIX_OP_MUL: acc(nd.a, g + " * " + B); acc(nd.b, g + " * " + A); break;
        case FELIX_OP_DIV: case FELIX_OP_FLOORDIV: case FELIX_OP_CEILDIV:
          o << "    const double t = " << g << " / " << B << ";\n";
          acc(nd.a, "t"); acc(nd.b, "t * " + V, true); break;
        case FELIX_OP_NEG: acc(nd.a, g, true); break;
        case FELIX_OP_POW: acc(nd.a, g + " * " + lit(nd.imm, true) + " * p_pow(" + A + ", " + lit(nd.imm - 1.0, true) + ")"); break;
        case FELIX_OP_EXP: acc(nd.a, g + " * " + V); break;
        case FELIX_OP_LOG: acc(nd.a, g + " / " + A); break;
        case FELIX_OP_SQRT: acc(nd.a, g + " * 0.5 / " + V); break;
        case FELIX_OP_MAX:
          o << "    const double s = sm_S(" << A << " - " << B << ");\n";
          acc(nd.a, g + " * s"); acc(nd.b, g + " * (1.0 - s)"); break;
        case FELIX_OP_MIN:
          o << "    const double s = sm_S(" << A << " - " << B << ");\n";
          acc(nd.a, g + " * (1.0 - s)"); acc(nd.b, g + " * s"); break;
        case FELIX_OP_GT: case FELIX_OP_GE:
          o << "    const double t = " << g << " * sm_dS(" << A << " - " << B << ");\n";
          acc(nd.a, "t"); acc(nd.b, "t", true); break;
        case FELIX_OP_LT: case FELIX_OP_LE:
          o << "    const double t = " << g << " * sm_dS(" << B << " - " << A << ");\n";
          acc(nd.a, "t", true); acc(nd.b, "t"); break;
        case FELIX_OP_EQ: case FELIX_OP_NE:
          o << "    const double dd = " << A << " - " << B << ";\n"
            << "    const double p = sm_S(dd + 0.5), q = sm_S(0.5 - dd);\n"
            << "    const double t = " << (nd.op == FELIX_OP_EQ ? "" : "-") << g << " * (sm_dS(dd + 0.5) * q - p * sm_dS(0.5 - dd));\n";
          acc(nd.a, "t"); acc(nd.b, "t", true); break;
        case FELIX_OP_AND: acc(nd.a, g + " * " + B); acc(nd.b, g + " * " + A); break;
        case FELIX_OP_OR: acc(nd.a, g + " * (1.0 - " + B + ")"); acc(nd.b, g + " * (1.0 - " + A + ")"); break;
        case FELIX_OP_NOT: acc(nd.a, g, true); break;
        case FELIX_OP_SELECT:
          acc(nd.a, g + " * (" + B + " - " + C + ")"); acc(nd.b, g + " * " + A); acc(nd.c, g + " * (1.0 - " + A + ")"); break;
        default: break;
      }
      o << "  }\n";
    }
  }
};

}  // namespace

int SpaceDesc::n_roots_total() const {
  int n_split = 0, n_int = 0;
  for (const auto& v : vars) (v.kind == FELIX_VAR_SPLIT ? n_split : n_int)++;
  return (int)croots.size() + n_split + (int)split_extent.size() + 2 * n_int;
}

std::string generate_dag_module(const SpaceDesc& d, int K0p, CodegenInfo* info) {
  Gen g(d);
  std::ostringstream& o = g.o;
  const int M = d.n_vars, K = (int)d.froots.size(), Ru = (int)d.croots.size();
  o << kPrelude;
  o << "#define NV " << M << "\n#define NF " << K << "\n#define NRU " << Ru << "\n#define NR " << d.n_roots_total()
    << "\n#define K0P " << K0p << "\n";

  // ---------------------------------------------------------------- automatic validity roots (y space)
  // emitted as a list of (value expr, [(var, +-1)]) for loss / seeds / gradient
  struct Auto { std::string val; std::vector<std::pair<int, int>> terms; };
  std::vector<Auto> autos;
  for (int j = 0; j < M; ++j)
    if (d.vars[j].kind == FELIX_VAR_SPLIT) autos.push_back({"-y" + std::to_string(j), {{j, -1}}});
  for (size_t s = 0; s < d.split_extent.size(); ++s) {
    std::string e = "(";
    std::vector<std::pair<int, int>> t;
    for (size_t k = 0; k < d.split_vars[s].size(); ++k) {
      int j = d.split_vars[s][k];
      e += (k ? " + y" : "y") + std::to_string(j);
      t.push_back({j, +1});
    }
    e += ") - " + lit(std::log((double)d.split_extent[s]), true);
    autos.push_back({e, t});
  }
  for (int j = 0; j < M; ++j)
    if (d.vars[j].kind == FELIX_VAR_INT) {
      autos.push_back({lit(std::log((double)d.vars[j].lo), true) + " - y" + std::to_string(j), {{j, -1}}});
      autos.push_back({"y" + std::to_string(j) + " - " + lit(std::log((double)d.vars[j].hi), true), {{j, +1}}});
    }

  // The smoothed DAG is evaluated in FP64 (forward and reverse): select chains whose branches differ
  // by ~1e5 amplify fp32 rounding of x - 1 beyond the 1e-4 feature tolerance.
  auto load_y = [&](const char* src) {
    for (int j = 0; j < M; ++j) o << "  const double y" << j << " = (double)" << src << "[(size_t)" << j << " * n + i];\n";
    for (int j = 0; j < M; ++j) o << "  const double x" << j << " = p_exp(y" << j << ");\n";
  };

  // ---------------------------------------------------------------- felix_fwd
  o << "extern \"C\" __global__ void __launch_bounds__(128) felix_fwd(const float* __restrict__ yv, int n, u16* __restrict__ phi_hi, u16* __restrict__ phi_lo) {\n"
    << "  const int i = blockIdx.x * blockDim.x + threadIdx.x;\n  if (i >= n) return;\n";
  load_y("yv");
  g.emit_forward(true, false, "x");
  const int64_t flops_fwd = g.flops;
  o << "  u32 ph[K0P / 2], pl[K0P / 2];\n";
  for (int k = 0; k < K0p; k += 2) {
    std::string f0 = k < K ? "(float)slogd_(v" + std::to_string(d.froots[k]) + ")" : "0.f";
    std::string f1 = k + 1 < K ? "(float)slogd_(v" + std::to_string(d.froots[k + 1]) + ")" : "0.f";
    o << "  { const float f0 = " << f0 << ", f1 = " << f1 << "; const u16 h0 = f2h(f0), h1 = f2h(f1);\n"
      << "    ph[" << k / 2 << "] = (u32)h0 | ((u32)h1 << 16); pl[" << k / 2 << "] = (u32)f2h(f0 - h2f(h0)) | ((u32)f2h(f1 - h2f(h1)) << 16); }\n";
  }
  o << "  uint4* dh = reinterpret_cast<uint4*>(phi_hi + (size_t)i * K0P);\n"
    << "  uint4* dl = reinterpret_cast<uint4*>(phi_lo + (size_t)i * K0P);\n"
    << "#pragma unroll\n  for (int q = 0; q < K0P / 8; ++q) { dh[q] = make_uint4(ph[4*q], ph[4*q+1], ph[4*q+2], ph[4*q+3]); dl[q] = make_uint4(pl[4*q], pl[4*q+1], pl[4*q+2], pl[4*q+3]); }\n"
    << "}\n\n";

  // ---------------------------------------------------------------- felix_rev (template on mode)
  o << "template <int EVAL>\n__device__ __forceinline__ void rev_body(float* __restrict__ yv, const float* __restrict__ yin, int n,\n"
    << "    const float* __restrict__ dphi, int ld_dphi, const float* __restrict__ c_part, int n_head_tiles, int ld_c, float head_b, float lam,\n"
    << "    float* __restrict__ mv, float* __restrict__ vv, int t, float lr, float b1, float b2, float eps,\n"
    << "    float* __restrict__ o_phi, float* __restrict__ o_g, float* __restrict__ o_cost, float* __restrict__ o_loss, float* __restrict__ o_grad) {\n"
    << "  const int i = blockIdx.x * blockDim.x + threadIdx.x;\n  if (i >= n) return;\n";
  load_y("yin");
  g.emit_forward(true, false, "x");
  // cost, constraints, loss
  o << "  float c = head_b;\n  for (int q = 0; q < n_head_tiles; ++q) c += c_part[(size_t)q * ld_c + i];\n";
  o << "  double pen = 0.0;\n";
  for (int r = 0; r < Ru; ++r) {
    o << "  const double g" << r << " = v" << d.croots[r] << "; const double p" << r << " = fmax(g" << r << ", 0.0); pen += p" << r << " * p" << r << ";\n";
  }
  for (size_t q = 0; q < autos.size(); ++q) {
    int r = Ru + (int)q;
    o << "  const double g" << r << " = " << autos[q].val << "; const double p" << r << " = fmax(g" << r << ", 0.0); pen += p" << r << " * p" << r << ";\n";
  }
  o << "  const float loss = (float)(-(double)c + (double)lam * pen);\n";
  // seeds
  g.emit_reverse();
  auto adj_name = [&](int node) {
    return d.nodes[node].op == FELIX_OP_VAR ? "gx" + std::to_string((int)d.nodes[node].imm) : "a" + std::to_string(node);
  };
  for (int k = 0; k < K; ++k) {
    int r = d.froots[k];
    if (!g.depvar[r]) continue;
    o << "  " << adj_name(r) << " += (double)dphi[(size_t)" << k << " * ld_dphi + i] * slogpd_(v" << r << ");\n";
  }
  for (int r = 0; r < Ru; ++r) {
    int nd = d.croots[r];
    if (!g.depvar[nd]) continue;
    o << "  " << adj_name(nd) << " += 2.0 * (double)lam * p" << r << ";\n";
  }
  g.emit_reverse_body();
  // dL/dy = x * adj(x) + auto-root terms
  for (int j = 0; j < M; ++j) o << "  double gd" << j << " = x" << j << " * gx" << j << ";\n";
  for (size_t q = 0; q < autos.size(); ++q) {
    int r = Ru + (int)q;
    for (auto& tv : autos[q].terms)
      o << "  gd" << tv.first << (tv.second > 0 ? " += " : " -= ") << "2.0 * (double)lam * p" << r << ";\n";
  }
  for (int j = 0; j < M; ++j) o << "  const float gy" << j << " = (float)gd" << j << ";\n";
  o << "  if (EVAL) {\n";
  o << "    if (o_phi) {\n";
  for (int k = 0; k < K; ++k) o << "      o_phi[(size_t)" << k << " * n + i] = (float)slogd_(v" << d.froots[k] << ");\n";
  o << "    }\n    if (o_g) {\n";
  for (int r = 0; r < d.n_roots_total(); ++r) o << "      o_g[(size_t)" << r << " * n + i] = (float)g" << r << ";\n";
  o << "    }\n    if (o_cost) o_cost[i] = c;\n    if (o_loss) o_loss[i] = loss;\n    if (o_grad) {\n";
  for (int j = 0; j < M; ++j) o << "      o_grad[(size_t)" << j << " * n + i] = gy" << j << ";\n";
  o << "    }\n  } else {\n";
  o << "    if (o_loss) o_loss[i] = loss;\n";
  o << "    bool ok = isfinite(loss)";
  for (int j = 0; j < M; ++j) o << " && isfinite(gy" << j << ")";
  o << ";\n    if (ok) {\n"
    << "      const float bc1 = 1.f - powf(b1, (float)t), bc2 = 1.f - powf(b2, (float)t);\n"
    << "      const float step = lr / bc1, rb = 1.f / sqrtf(bc2);\n";
  for (int j = 0; j < M; ++j) {
    o << "      { const size_t o_ = (size_t)" << j << " * n + i; float m = mv[o_], v = vv[o_];\n"
      << "        m = b1 * m + (1.f - b1) * gy" << j << "; v = b2 * v + (1.f - b2) * gy" << j << " * gy" << j << ";\n"
      << "        mv[o_] = m; vv[o_] = v; yv[o_] = y" << j << " - step * m / (sqrtf(v) * rb + eps); }\n";
  }
  o << "    }\n  }\n}\n\n";
  o << "extern \"C\" __global__ void __launch_bounds__(128) felix_rev_adam(float* yv, int n, const float* dphi, int ld_dphi, const float* c_part, int n_head_tiles, int ld_c, float head_b, float lam,\n"
    << "    float* mv, float* vv, int t, float lr, float b1, float b2, float eps, float* o_loss) {\n"
    << "  rev_body<0>(yv, yv, n, dphi, ld_dphi, c_part, n_head_tiles, ld_c, head_b, lam, mv, vv, t, lr, b1, b2, eps, nullptr, nullptr, nullptr, o_loss, nullptr);\n}\n";
  o << "extern \"C\" __global__ void __launch_bounds__(128) felix_rev_eval(const float* yv, int n, const float* dphi, int ld_dphi, const float* c_part, int n_head_tiles, int ld_c, float head_b, float lam,\n"
    << "    float* o_phi, float* o_g, float* o_cost, float* o_loss, float* o_grad) {\n"
    << "  rev_body<1>(nullptr, yv, n, dphi, ld_dphi, c_part, n_head_tiles, ld_c, head_b, lam, nullptr, nullptr, 0, 0.f, 0.f, 0.f, 0.f, o_phi, o_g, o_cost, o_loss, o_grad);\n}\n\n";

  // ---------------------------------------------------------------- felix_hard (fp64, integer points)
  o << "extern \"C\" __global__ void __launch_bounds__(128) felix_hard(const int* __restrict__ sched, int n, double* __restrict__ phi64, unsigned char* __restrict__ valid) {\n"
    << "  const int i = blockIdx.x * blockDim.x + threadIdx.x;\n  if (i >= n) return;\n";
  for (int j = 0; j < M; ++j) o << "  const double h" << j << " = (double)sched[(size_t)i * NV + " << j << "];\n";
  g.emit_forward(true, true, "h");
  o << "  bool ok = true;\n";
  for (int k = 0; k < K; ++k)
    o << "  ok = ok && isfinite(v" << d.froots[k] << "); phi64[(size_t)" << k << " * n + i] = slogd_(v" << d.froots[k] << ");\n";
  for (int r = 0; r < Ru; ++r) o << "  ok = ok && isfinite(v" << d.croots[r] << ") && (v" << d.croots[r] << " <= 1e-9);\n";
  o << "  valid[i] = ok ? 1 : 0;\n}\n\n";

  // ---------------------------------------------------------------- felix_init (rejection sampler)
  // components of the var-split incidence graph (same construction as the rounding tables)
  std::vector<int> parent(M);
  for (int j = 0; j < M; ++j) parent[j] = j;
  std::function<int(int)> find = [&](int j) { while (parent[j] != j) { parent[j] = parent[parent[j]]; j = parent[j]; } return j; };
  for (auto& sv : d.split_vars) for (size_t k = 1; k < sv.size(); ++k) parent[find(sv[k])] = find(sv[0]);
  std::vector<std::vector<int>> comps;
  {
    std::vector<int> root_of(M, -1);
    for (int j = 0; j < M; ++j) {
      if (d.vars[j].kind != FELIX_VAR_SPLIT) continue;
      int r = find(j);
      if (root_of[r] < 0) { root_of[r] = (int)comps.size(); comps.push_back({}); }
      comps[root_of[r]].push_back(j);
    }
  }
  o << "extern \"C\" __global__ void __launch_bounds__(128) felix_init(u64 seed, int n, long long index_base, float* __restrict__ yout) {\n"
    << "  const int i = blockIdx.x * blockDim.x + threadIdx.x;\n  if (i >= n) return;\n"
    << "  const u64 cand = (u64)(index_base + i);\n";
  for (int j = 0; j < M; ++j) o << "  double y" << j << " = 0.0;\n";
  o << "  bool done = false;\n  for (int a2 = 0; a2 < 64 && !done; ++a2) {\n";
  for (size_t ci = 0; ci < comps.size(); ++ci) {
    const auto& comp = comps[ci];
    o << "    {\n      bool acc = false;\n";
    for (int j : comp) o << "      double c" << j << " = 0.0;\n";
    o << "      for (int a1 = 0; a1 < 64 && !acc; ++a1) {\n        const u64 att = (u64)(a2 * 64 + a1);\n";
    for (int j : comp) {
      double ub = 1e300;
      for (size_t s = 0; s < d.split_vars.size(); ++s)
        for (int v : d.split_vars[s]) if (v == j) ub = std::min(ub, (double)d.split_extent[s]);
      o << "        const double t" << j << " = __dmul_rn(cuni(seed, cand, att, " << j << "ull), " << lit(std::log(ub), true) << ");\n";
    }
    o << "        bool ok = true;\n";
    for (size_t s = 0; s < d.split_vars.size(); ++s) {
      bool mine = false;
      for (int v : d.split_vars[s]) for (int j : comp) if (v == j) mine = true;
      if (!mine) continue;
      o << "        { double tot = 0.0;";
      for (int v : d.split_vars[s]) o << " tot = __dadd_rn(tot, t" << v << ");";
      o << " ok = ok && (__dsub_rn(tot, " << lit(std::log((double)d.split_extent[s]), true) << ") <= 0.0); }\n";
    }
    o << "        if (ok) { acc = true;";
    for (int j : comp) o << " c" << j << " = t" << j << ";";
    o << " }\n      }\n";
    for (int j : comp) o << "      y" << j << " = c" << j << ";\n";
    o << "    }\n";
  }
  for (int j = 0; j < M; ++j) {
    if (d.vars[j].kind != FELIX_VAR_INT) continue;
    double llo = std::log((double)d.vars[j].lo), lhi = std::log((double)d.vars[j].hi);
    o << "    y" << j << " = __dadd_rn(" << lit(llo, true) << ", __dmul_rn(cuni(seed, cand, (u64)(a2 * 64), " << j << "ull), "
      << lit(lhi - llo, true) << "));\n";
  }
  o << "    {\n";
  for (int j = 0; j < M; ++j) o << "      const double x" << j << " = exp(y" << j << ");\n";
  // fp64 smooth forward (only constraint roots are used; dead code is eliminated)
  {
    std::ostringstream save;
    save << o.str();
    o.str(""); o.clear();
    g.emit_forward(true, false, "x");
    std::string body = o.str();
    o.str(""); o.clear();
    o << save.str();
    std::istringstream in(body);
    std::string line;
    while (std::getline(in, line)) o << "    " << line << "\n";
  }
  o << "      bool ok = true;\n";
  for (int r = 0; r < Ru; ++r) o << "      ok = ok && (v" << d.croots[r] << " <= 0.0);\n";
  o << "      if (ok) done = true;\n    }\n  }\n  if (!done) {\n";
  for (int j = 0; j < M; ++j)
    o << "    y" << j << " = " << (d.vars[j].kind == FELIX_VAR_INT ? lit(std::log((double)d.vars[j].lo), true) : "0.0") << ";\n";
  o << "  }\n";
  for (int j = 0; j < M; ++j) o << "  yout[(size_t)" << j << " * n + i] = (float)y" << j << ";\n";
  o << "}\n";

  if (info) info->flops_fwd = flops_fwd;
  return o.str();
}

}  // namespace felix
