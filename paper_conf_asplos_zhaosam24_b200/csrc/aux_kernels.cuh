// aux_kernels.cuh — rounding, FP64 scoring and top-k (Algorithm 1 lines 20-21, P:L919-920,
// P:L928-935).  All decisions that produce integers are taken in FP64 with explicitly rounded
// operations (no FMA contraction) against host-built ln tables, so they are reproducible
// bit-for-bit by the float64 oracle (DESIGN.md "Readings" O10, R-valid).
#pragma once
#include <cstdint>
#include <cfloat>

namespace felix {

// ---------------------------------------------------------------------------- K5a split rounding
// One warp per (candidate, split component): lanes stride over the component's divisor-tuple
// table (lexicographic order) computing sum_j (y_j - ln f_j)^2; warp argmin, ties -> lower index
// (= lexicographically smallest tuple).  Reading O10 of P:L796-801 ("rounds y to the closest ln N_i").
__global__ void __launch_bounds__(256) round_split_kernel(
    const float* __restrict__ y, int n, int M, int n_comp,
    const int* __restrict__ comp_nvars, const int* __restrict__ comp_var0, const int* __restrict__ comp_vars,
    const long long* __restrict__ comp_eoff, const long long* __restrict__ comp_tcount,
    const int* __restrict__ tuples, const double* __restrict__ lnf, int* __restrict__ sched) {
  const long long gw = (static_cast<long long>(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (gw >= static_cast<long long>(n) * n_comp) return;
  const int cand = static_cast<int>(gw / n_comp), comp = static_cast<int>(gw % n_comp);
  const int nv = comp_nvars[comp];
  const int* vars = comp_vars + comp_var0[comp];
  double yv[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) yv[k] = k < nv ? static_cast<double>(y[static_cast<size_t>(vars[k]) * n + cand]) : 0.0;
  const long long eoff = comp_eoff[comp], T = comp_tcount[comp];
  if (T < 0) return;                               // no table: round_bnb_kernel searches this component
  double best = DBL_MAX;
  long long bi = -1;
  for (long long t = lane; t < T; t += 32) {
    const double* l = lnf + eoff + t * nv;
    double acc = 0.0;
    for (int k = 0; k < nv; ++k) {
      const double d = __dsub_rn(yv[k], l[k]);
      acc = __dadd_rn(acc, __dmul_rn(d, d));
    }
    if (acc < best) { best = acc; bi = t; }     // strict: first minimum in this lane's stride
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    const double ob = __shfl_xor_sync(0xffffffffu, best, off);
    const long long oi = __shfl_xor_sync(0xffffffffu, bi, off);
    const bool take = (oi >= 0) && (bi < 0 || ob < best || (ob == best && oi < bi));
    if (take) { best = ob; bi = oi; }
  }
  if (lane == 0) {
    if (bi < 0) bi = 0;    // all distances NaN: first tuple (all ones), as np.argmin
    const int* tp = tuples + eoff + bi * nv;
    for (int k = 0; k < nv; ++k) sched[static_cast<size_t>(cand) * M + vars[k]] = tp[k];
  }
}

// ---------------------------------------------------------------------------- K5a' branch and bound
// The same argmin as round_split_kernel (sum_j (y_j - ln f_j)^2 over the divisor-respecting tuples,
// FP64 in var order, explicitly rounded, ties -> lexicographically smallest tuple) for components whose
// tuple table would be too large (highly composite extents, SURVEY §7c hard part 7; N is
// "typically smaller than 10^6", and 720720 split four ways has 6.6e5 tuples, eight ways 1.5e8).
// One thread per (candidate, component): depth-first over the component's vars in order; at depth k
// the divisors of the var's gcd extent are visited outward from y_k (nearest first), a divisor is
// taken only if it divides every remaining split extent the var belongs to, and a direction stops
// as soon as partial + (y_k - ln d)^2 > best: the remaining terms are >= 0 and FP64 addition is
// monotone, so every pruned tuple costs strictly more than the best found.  A child is also skipped
// when partial + LB > best, LB a lower bound of the remaining vars' cost under the product constraint
// (ln f_j >= 0 and sum_{j in split q} ln f_j <= ln rem_q): per var (y_j < 0: y_j^2; y_j > ln rem: the
// excess squared), and per split (sum of the positive y_j - ln rem_q)^2 / (their count) by Cauchy-Schwarz;
// compared with a 1e-9 relative margin, far above the FP64 rounding of the leaf sums (~1e-15), so a
// skipped subtree never holds a tuple that ties or beats the best.  Without it an eight-way split of
// 720720 visits most of its 1.5e8 tuples.  Leaves replace the best
// on a smaller cost or on an equal cost and a lexicographically smaller tuple, so the result is the
// exhaustive scan's bit for bit.  Non-finite y anywhere in the component: every tuple costs inf / NaN
// and the scan returns its first tuple, all ones; so does this kernel.
// Exact lower bound for single-split components (every var tiles the same extent E): one warp per
// (candidate, component) first fills V[k][r] = min over f | r of (y_k - ln f)^2 + V[k+1][r / f] (V[nv] = 0,
// r over the divisors of E: the cost of vars k .. nv-1 when their product must divide r, a dynamic
// programme over the remaining extent) in shared memory, lanes over r.  Lane 0 then takes the DP's own
// argmin path as the first incumbent and runs the search above with the child test
// (partial + (y_k - ln d)^2 + V[k+1][rem / d]) * (1 - 1e-12) > best: V is the exact optimum of the
// remaining vars up to FP64 rounding (~1e-15 relative), so only near-ties of the best are visited and the
// leaves -- summed left to right exactly as the table scan sums them -- decide, bit for bit.
// Components touching several splits (or whose table would not fit) use the weaker bound above.
__device__ __forceinline__ int bnb_div_index(const long long* __restrict__ D, int cnt, long long x) {
  int a = 0, b = cnt - 1;
  while (a < b) { const int m = (a + b) >> 1; if (D[m] < x) a = m + 1; else b = m; }
  return a;
}

__global__ void __launch_bounds__(128) round_bnb_kernel(
    const float* __restrict__ y, int n, int M, int n_sel, const int* __restrict__ sel_comp,
    const int* __restrict__ comp_nvars, const int* __restrict__ comp_var0, const int* __restrict__ comp_vars,
    const int* __restrict__ comp_ns, const int* __restrict__ comp_s0, const long long* __restrict__ comp_sext,
    const unsigned* __restrict__ var_smask, const long long* __restrict__ var_doff, const int* __restrict__ var_dcnt,
    const long long* __restrict__ dval, const double* __restrict__ dln, int* __restrict__ sched, int dp_cap) {
  extern __shared__ double bnb_smem[];
  const long long g = (static_cast<long long>(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;   // warp per item
  const int lane = threadIdx.x & 31;
  if (g >= static_cast<long long>(n) * n_sel) return;
  double* V = bnb_smem + (threadIdx.x >> 5) * (dp_cap / 8);
  const int cand = static_cast<int>(g / n_sel), comp = sel_comp[g % n_sel];
  const int nv = comp_nvars[comp], v0 = comp_var0[comp], ns = comp_ns[comp];
  const int* vars = comp_vars + v0;
  double yv[8];
  bool finite = true;
  for (int k = 0; k < nv; ++k) {
    yv[k] = static_cast<double>(y[static_cast<size_t>(vars[k]) * n + cand]);
    finite = finite && isfinite(yv[k]);
  }
  // the DP bound: one split, every var's divisor list = the divisors of E
  const int nd = var_dcnt[v0];
  const bool dp = finite && ns == 1 && (nv + 1) * nd * 8 <= dp_cap;
  const long long* DE = dval + var_doff[v0];
  const double* LE = dln + var_doff[v0];
  if (dp) {
    for (int i = lane; i < nd; i += 32) V[nv * nd + i] = 0.0;
    __syncwarp();
    for (int k = nv - 1; k >= 0; --k) {
      for (int i = lane; i < nd; i += 32) {
        const long long r = DE[i];
        double m = DBL_MAX;
        for (int j = 0; j <= i; ++j) {
          if (r % DE[j] != 0) continue;
          const double d = yv[k] - LE[j];
          m = fmin(m, d * d + V[(k + 1) * nd + bnb_div_index(DE, nd, r / DE[j])]);
        }
        V[k * nd + i] = m;
      }
      __syncwarp();
    }
  }
  if (lane != 0) return;
  long long bt[8];
  for (int k = 0; k < nv; ++k) bt[k] = 1;
  if (finite) {
    long long rem[16];
    for (int q = 0; q < ns; ++q) rem[q] = comp_sext[comp_s0[comp] + q];
    int lo[8], hi[8];
    double acc[9];
    long long cur[8];
    double best = DBL_MAX;
    bool found = false;
    if (dp) {
      // incumbent: the DP's argmin path (ties -> smallest divisor), its cost summed as the leaves are
      long long r = rem[0];
      double c = 0.0;
      for (int k = 0; k < nv; ++k) {
        const int ir = bnb_div_index(DE, nd, r);
        double m = DBL_MAX;
        long long fb = 1;
        for (int j = 0; j <= ir; ++j) {
          if (r % DE[j] != 0) continue;
          const double d = yv[k] - LE[j];
          const double v = d * d + V[(k + 1) * nd + bnb_div_index(DE, nd, r / DE[j])];
          if (v < m) { m = v; fb = DE[j]; }
        }
        bt[k] = fb;
        r /= fb;
      }
      for (int k = 0; k < nv; ++k) {
        const double d = __dsub_rn(yv[k], LE[bnb_div_index(DE, nd, bt[k])]);
        c = __dadd_rn(c, __dmul_rn(d, d));
      }
      best = c;
      found = true;
    }
    // position of y_k among the ascending ln d of var k: lo = last index with ln d < y, hi = lo + 1
    auto start = [&](int k) {
      const double* L = dln + var_doff[v0 + k];
      int a = 0, b = var_dcnt[v0 + k];
      while (a < b) { const int m = (a + b) >> 1; if (L[m] < yv[k]) a = m + 1; else b = m; }
      lo[k] = a - 1; hi[k] = a;
    };
    acc[0] = 0.0;
    int k = 0;
    start(0);
    while (k >= 0) {
      const double* L = dln + var_doff[v0 + k];
      const long long* D = dval + var_doff[v0 + k];
      const int cnt = var_dcnt[v0 + k];
      double elo = DBL_MAX, ehi = DBL_MAX;
      bool olo = false, ohi = false;
      if (lo[k] >= 0) {
        const double d = __dsub_rn(yv[k], L[lo[k]]);
        elo = __dadd_rn(acc[k], __dmul_rn(d, d));
        olo = !(elo > best);
      }
      if (hi[k] < cnt) {
        const double d = __dsub_rn(yv[k], L[hi[k]]);
        ehi = __dadd_rn(acc[k], __dmul_rn(d, d));
        ohi = !(ehi > best);
      }
      if (!olo && !ohi) {                       // level exhausted: back up, restoring the extents
        --k;
        if (k >= 0) {
          const unsigned msk = var_smask[v0 + k];
          for (int q = 0; q < ns; ++q) if (msk >> q & 1u) rem[q] *= cur[k];
        }
        continue;
      }
      const bool take_lo = olo && (!ohi || elo <= ehi);
      const int idx = take_lo ? lo[k]-- : hi[k]++;
      const double e = take_lo ? elo : ehi;
      const long long dv = D[idx];
      const unsigned msk = var_smask[v0 + k];
      bool ok = true;
      for (int q = 0; q < ns; ++q) if ((msk >> q & 1u) && rem[q] % dv != 0) ok = false;
      if (!ok) continue;
      if (k == nv - 1) {                        // leaf
        bool better = !found || e < best;
        if (!better && e == best) {
          cur[k] = dv;
          int q = 0;
          while (q < nv && cur[q] == bt[q]) ++q;
          better = q < nv && cur[q] < bt[q];
        }
        if (better) {
          best = e; found = true;
          cur[k] = dv;
          for (int q = 0; q < nv; ++q) bt[q] = cur[q];
        }
        continue;
      }
      cur[k] = dv;
      for (int q = 0; q < ns; ++q) if (msk >> q & 1u) rem[q] /= dv;
      double lb;
      if (dp) {
        lb = V[(k + 1) * nd + bnb_div_index(DE, nd, rem[0])];
      } else {
        // lower bound of the cost of vars k+1 .. nv-1 under the remaining extents
        double lnr[16];
        for (int q = 0; q < ns; ++q) lnr[q] = log(static_cast<double>(rem[q]));
        double lb_var = 0.0, lb_neg = 0.0, lb_split = 0.0;
        double psum[16];
        int pcnt[16];
        for (int q = 0; q < ns; ++q) { psum[q] = 0.0; pcnt[q] = 0; }
        for (int j = k + 1; j < nv; ++j) {
          const unsigned mj = var_smask[v0 + j];
          const double yj = yv[j];
          if (yj < 0.0) { lb_neg += yj * yj; continue; }
          double cap = DBL_MAX;
          for (int q = 0; q < ns; ++q)
            if (mj >> q & 1u) { cap = fmin(cap, lnr[q]); psum[q] += yj; pcnt[q] += 1; }
          if (yj > cap) lb_var += (yj - cap) * (yj - cap);
        }
        for (int q = 0; q < ns; ++q) {
          const double ex = psum[q] - lnr[q];
          if (pcnt[q] > 0 && ex > 0.0) lb_split = fmax(lb_split, ex * ex / pcnt[q]);
        }
        lb = fmax(lb_neg + lb_var, lb_neg + lb_split);
      }
      if ((e + lb) * (1.0 - 1e-9) > best) {     // nothing below this child can tie or beat the best
        for (int q = 0; q < ns; ++q) if (msk >> q & 1u) rem[q] *= dv;
        continue;
      }
      acc[k + 1] = e;
      ++k;
      start(k);
    }
  }
  for (int k = 0; k < nv; ++k) sched[static_cast<size_t>(cand) * M + vars[k]] = static_cast<int>(bt[k]);
}

// ---------------------------------------------------------------------------- K5b INT rounding
// x = lo + #{k in [lo, hi-1] : ln(k + 1/2) <= y}  (nearest integer), binary search.
__global__ void round_int_kernel(const float* __restrict__ y, int n, int M, int n_int, const int* __restrict__ int_vars,
                                 const long long* __restrict__ int_lo, const long long* __restrict__ int_cnt,
                                 const long long* __restrict__ int_toff, const double* __restrict__ thr, int* __restrict__ sched) {
  const long long g = static_cast<long long>(blockIdx.x) * blockDim.x + threadIdx.x;
  if (g >= static_cast<long long>(n) * n_int) return;
  const int cand = static_cast<int>(g / n_int), q = static_cast<int>(g % n_int);
  const int j = int_vars[q];
  const double yv = static_cast<double>(y[static_cast<size_t>(j) * n + cand]);
  const double* t = thr + int_toff[q];
  long long lo = 0, hi = int_cnt[q];          // count of thresholds <= yv
  while (lo < hi) {
    const long long mid = (lo + hi) >> 1;
    if (t[mid] <= yv) lo = mid + 1; else hi = mid;
  }
  sched[static_cast<size_t>(cand) * M + j] = static_cast<int>(int_lo[q] + lo);
}

// ---------------------------------------------------------------------------- K6 FP64 MLP scoring
// out[row][col] = act( b[col] + sum_k W[col][k] * in(row, k) ), k ascending (deterministic, so equal
// schedules get bit-identical scores); accumulate != 0 adds to out (segment sum over statements).  32x32 output tile per 256-thread block, K staged through
// shared memory in chunks of 32; thread (tx, ty) owns column tx and rows ty*4 .. ty*4+3.
__global__ void __launch_bounds__(256) score_layer_kernel(const double* __restrict__ in, long long in_rs, long long in_cs,
                                                          int n, int K, const double* __restrict__ W,
                                                          const double* __restrict__ b, double* __restrict__ out,
                                                          int N, int relu, int accumulate) {
  __shared__ double As[32][33];   // [k][row]
  __shared__ double Bs[32][33];   // [k][col]
  const int tx = threadIdx.x, ty = threadIdx.y, tid = ty * 32 + tx;
  const int row0 = blockIdx.y * 32, col0 = blockIdx.x * 32;
  const int col = col0 + tx;
  double acc[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) acc[q] = (col < N) ? b[col] : 0.0;
  for (int k0 = 0; k0 < K; k0 += 32) {
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int e = tid + q * 256;           // 1024 elements of each 32x32 tile
      const int r = e & 31, kk = e >> 5;      // A: consecutive threads -> consecutive rows (SoA input)
      const int gr = row0 + r, gk = k0 + kk;
      As[kk][r] = (gr < n && gk < K) ? in[static_cast<size_t>(gr) * in_rs + static_cast<size_t>(gk) * in_cs] : 0.0;
      const int c = e >> 5, kb = e & 31;      // B: consecutive threads -> consecutive k (row-major W)
      const int gc = col0 + c, gkb = k0 + kb;
      Bs[kb][c] = (gc < N && gkb < K) ? W[static_cast<size_t>(gc) * K + gkb] : 0.0;
    }
    __syncthreads();
    const int kmax = min(32, K - k0);
    for (int kk = 0; kk < kmax; ++kk) {
      const double w = Bs[kk][tx];
#pragma unroll
      for (int q = 0; q < 4; ++q) acc[q] = fma(w, As[kk][ty * 4 + q], acc[q]);
    }
    __syncthreads();
  }
  if (col < N) {
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int r = row0 + ty * 4 + q;
      if (r < n) {
        const double v = (relu && !(acc[q] > 0.0)) ? 0.0 : acc[q];
        out[static_cast<size_t>(r) * N + col] = accumulate ? out[static_cast<size_t>(r) * N + col] + v : v;
      }
    }
  }
}

// ---------------------------------------------------------------------------- K6 FP64 MLP scoring (v2)
// Same arithmetic again (acc = b[col]; k ascending: acc = fma(W[col][k], in(row, k), acc)), bit-identical
// to the kernels above.  128 x 64 output tile per 256-thread block; thread (tx, ty) owns rows ty * 8 + i
// (i < 8) and 4 columns, 32 FP64 accumulators: per k, 4 + 2 16-byte shared loads (6 wavefronts per warp)
// feed 32 DFMA.  K is staged 16 at a
// time through double-buffered shared memory filled one chunk ahead from registers, one barrier per chunk.
constexpr int SC2_TM = 128, SC2_TN = 64, SC2_KT = 16;
__global__ void __launch_bounds__(256) score_layer_v2_kernel(const double* __restrict__ in, long long in_rs, long long in_cs,
                                                             int n, int K, const double* __restrict__ W,
                                                             const double* __restrict__ b, double* __restrict__ out,
                                                             int N, int relu, int accumulate) {
  __shared__ __align__(16) double As[2][SC2_KT][SC2_TM];   // [buf][k][row]
  __shared__ __align__(16) double Bs[2][SC2_KT][SC2_TN];   // [buf][k][col]
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  const int row0 = blockIdx.y * SC2_TM, col0 = blockIdx.x * SC2_TN;
  double acc[8][4];
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const int col = col0 + (j < 2 ? 2 * tx + j : 32 + 2 * tx + (j - 2));
    const double bj = col < N ? b[col] : 0.0;
#pragma unroll
    for (int i = 0; i < 8; ++i) acc[i][j] = bj;
  }
  // per chunk: A tile 16 x 128 (8 per thread), W tile 16 x 64 (4 per thread)
  double pa[8], pb[4];
  auto load_chunk = [&](int k0) {
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const int e = tid + q * 256;
      int r, kk;
      if (in_rs == 1) { r = e & 127; kk = e >> 7; } else { kk = e & 15; r = e >> 4; }
      const int gr = row0 + r, gk = k0 + kk;
      pa[q] = (gr < n && gk < K) ? in[static_cast<size_t>(gr) * in_rs + static_cast<size_t>(gk) * in_cs] : 0.0;
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int e = tid + q * 256;
      const int c = e >> 4, kb = e & 15;
      const int gc = col0 + c, gkb = k0 + kb;
      pb[q] = (gc < N && gkb < K) ? W[static_cast<size_t>(gc) * K + gkb] : 0.0;
    }
  };
  auto store_chunk = [&](int buf) {
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const int e = tid + q * 256;
      int r, kk;
      if (in_rs == 1) { r = e & 127; kk = e >> 7; } else { kk = e & 15; r = e >> 4; }
      As[buf][kk][r] = pa[q];
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int e = tid + q * 256;
      Bs[buf][e & 15][e >> 4] = pb[q];
    }
  };
  const int nk = (K + SC2_KT - 1) / SC2_KT;
  load_chunk(0);
  store_chunk(0);
  __syncthreads();
  for (int c = 0; c < nk; ++c) {
    const int buf = c & 1;
    if (c + 1 < nk) load_chunk((c + 1) * SC2_KT);
    const int kmax = min(SC2_KT, K - c * SC2_KT);
    // thread (tx, ty): rows ty * 8 .. + 7 (4 x 16-B loads, two distinct addresses per warp: broadcast) and
    // columns 2 tx, 2 tx + 1, 32 + 2 tx, 33 + 2 tx (2 x 16-B loads over 256 consecutive bytes: 2 wavefronts)
    auto kstep = [&](int kk) {
      double a[8], w[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const double2 v = *reinterpret_cast<const double2*>(&As[buf][kk][ty * 8 + 2 * i]);
        a[2 * i] = v.x; a[2 * i + 1] = v.y;
      }
      const double2 w01 = *reinterpret_cast<const double2*>(&Bs[buf][kk][2 * tx]);
      const double2 w23 = *reinterpret_cast<const double2*>(&Bs[buf][kk][32 + 2 * tx]);
      w[0] = w01.x; w[1] = w01.y; w[2] = w23.x; w[3] = w23.y;
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fma(w[j], a[i], acc[i][j]);
    };
    if (kmax == SC2_KT) {
#pragma unroll
      for (int kk = 0; kk < SC2_KT; ++kk) kstep(kk);
    } else {
      for (int kk = 0; kk < kmax; ++kk) kstep(kk);
    }
    if (c + 1 < nk) store_chunk(buf ^ 1);   // the other buffer was last read in chunk c - 1 (barrier below)
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = row0 + ty * 8 + i;
    if (r >= n) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int col = col0 + (j < 2 ? 2 * tx + j : 32 + 2 * tx + (j - 2));
      if (col >= N) continue;
      const double v = (relu && !(acc[i][j] > 0.0)) ? 0.0 : acc[i][j];
      out[static_cast<size_t>(r) * N + col] = accumulate ? out[static_cast<size_t>(r) * N + col] + v : v;
    }
  }
}

// The same layer on the FP64 tensor cores (mma.sync m8n8k4 f64): 128 x 64 tiles, 8 warps of 32 x 32 (4 x 4
// MMAs of 8 x 8 per K step of 4, 32 accumulators per thread), K staged 16 at a time through double-buffered
// shared memory (rows padded so a fragment load of 4 k x 8 doubles takes the minimum two wavefronts).  Each
// thread's fragment loads feed 2 MMAs per load instead of the CUDA-core kernel's 32 DFMA per 6 loads at one
// CTA per SM; FP64 throughout, products summed by the MMA unit (differences to the CUDA-core order are at
// the 1e-16 level, far inside the 1e-12 score tolerance).
// MI = 8-row MMA blocks per warp tile: 4 (128 x 64 block tiles, 32 x 32 warp tiles) or 8 (256 x 64 block
// tiles, 64 x 32 warp tiles: 12 fragment loads per 32 MMAs instead of 8 per 16; used when the population
// gives at least two such tiles per SM).
constexpr int SCD_TN = 64, SCD_KT = 16, SCD_BP = SCD_TN + 4;
template <int MI> __host__ __device__ constexpr int scd_tm() { return 32 * MI; }
template <int MI> __host__ __device__ constexpr int scd_ap() { return 32 * MI + 4; }
template <int MI> __host__ __device__ constexpr int scd_smem() { return 2 * SCD_KT * (scd_ap<MI>() + SCD_BP) * 8; }   // dynamic, opt-in
template <int MI>
__global__ void __launch_bounds__(256, MI == 4 ? 2 : 1) score_layer_dmma_kernel(const double* __restrict__ in, long long in_rs, long long in_cs,
                                                               int n, int K, const double* __restrict__ W,
                                                               const double* __restrict__ b, double* __restrict__ out,
                                                               int N, int relu, int accumulate) {
  extern __shared__ __align__(16) double scd_smem[];
  constexpr int TM = scd_tm<MI>(), AP = scd_ap<MI>();
  double (*As)[SCD_KT][AP] = reinterpret_cast<double (*)[SCD_KT][AP]>(scd_smem);                      // [buf][k][row]
  double (*Bs)[SCD_KT][SCD_BP] = reinterpret_cast<double (*)[SCD_KT][SCD_BP]>(scd_smem + 2 * SCD_KT * AP);  // [buf][k][col]
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int gid = lane >> 2, tig = lane & 3;
  const int wr = (warp & 3) * (8 * MI), wc = (warp >> 2) * 32;    // warp tile origin inside the block tile
  const int row0 = blockIdx.y * TM, col0 = blockIdx.x * SCD_TN;
  double acc[MI][4][2];
#pragma unroll
  for (int nj = 0; nj < 4; ++nj) {
    const int c = col0 + wc + nj * 8 + 2 * tig;
    const double b0 = c < N ? b[c] : 0.0, b1 = c + 1 < N ? b[c + 1] : 0.0;
#pragma unroll
    for (int mi = 0; mi < MI; ++mi) { acc[mi][nj][0] = b0; acc[mi][nj][1] = b1; }
  }
  constexpr int QA = TM * SCD_KT / 256;   // A elements per thread per chunk
  double pa[QA], pb[4];
  auto load_chunk = [&](int k0) {
#pragma unroll
    for (int q = 0; q < QA; ++q) {
      const int e = tid + q * 256;
      int r, kk;
      if (in_rs == 1) { r = e % TM; kk = e / TM; } else { kk = e & 15; r = e >> 4; }
      const int gr = row0 + r, gk = k0 + kk;
      pa[q] = (gr < n && gk < K) ? in[static_cast<size_t>(gr) * in_rs + static_cast<size_t>(gk) * in_cs] : 0.0;
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int e = tid + q * 256;
      const int c = e >> 4, kb = e & 15;
      const int gc = col0 + c, gkb = k0 + kb;
      pb[q] = (gc < N && gkb < K) ? W[static_cast<size_t>(gc) * K + gkb] : 0.0;
    }
  };
  auto store_chunk = [&](int buf) {
#pragma unroll
    for (int q = 0; q < QA; ++q) {
      const int e = tid + q * 256;
      int r, kk;
      if (in_rs == 1) { r = e % TM; kk = e / TM; } else { kk = e & 15; r = e >> 4; }
      As[buf][kk][r] = pa[q];
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int e = tid + q * 256;
      Bs[buf][e & 15][e >> 4] = pb[q];
    }
  };
  const int nk = (K + SCD_KT - 1) / SCD_KT;
  load_chunk(0);
  store_chunk(0);
  __syncthreads();
  for (int c = 0; c < nk; ++c) {
    const int buf = c & 1;
    if (c + 1 < nk) load_chunk((c + 1) * SCD_KT);
    // zero-padded K: the chunk's k beyond K are 0 in both operands, so all 4 K steps run
#pragma unroll
    for (int k4 = 0; k4 < SCD_KT; k4 += 4) {
      double af[MI], bf[4];
#pragma unroll
      for (int mi = 0; mi < MI; ++mi) af[mi] = As[buf][k4 + tig][wr + mi * 8 + gid];
#pragma unroll
      for (int nj = 0; nj < 4; ++nj) bf[nj] = Bs[buf][k4 + tig][wc + nj * 8 + gid];
#pragma unroll
      for (int mi = 0; mi < MI; ++mi)
#pragma unroll
        for (int nj = 0; nj < 4; ++nj)
          asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};"
                       : "+d"(acc[mi][nj][0]), "+d"(acc[mi][nj][1]) : "d"(af[mi]), "d"(bf[nj]));
    }
    if (c + 1 < nk) store_chunk(buf ^ 1);   // the other buffer was last read in chunk c - 1 (barrier below)
    __syncthreads();
  }
#pragma unroll
  for (int mi = 0; mi < MI; ++mi) {
    const int r = row0 + wr + mi * 8 + gid;
    if (r >= n) continue;
#pragma unroll
    for (int nj = 0; nj < 4; ++nj) {
      const int col = col0 + wc + nj * 8 + 2 * tig;
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        if (col + h >= N) continue;
        const double v = (relu && !(acc[mi][nj][h] > 0.0)) ? 0.0 : acc[mi][nj][h];
        double* o = out + static_cast<size_t>(r) * N + col + h;
        *o = accumulate ? *o + v : v;
      }
    }
  }
}

// head layer (N = 1, row-major input [n][K]): thread per row streaming its own row (the L1 serves the
// 16 doubles of each 128-B line), one-warp blocks so the rows spread over the SMs; same fma order as above
__global__ void __launch_bounds__(32) score_head_kernel(const double* __restrict__ in, int n, int K,
                                                        const double* __restrict__ W, const double* __restrict__ b,
                                                        double* __restrict__ out, int accumulate) {
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= n) return;
  const double* __restrict__ row = in + static_cast<size_t>(r) * K;
  double acc = b[0];
#pragma unroll 8
  for (int k = 0; k < K; ++k) acc = fma(W[k], row[k], acc);
  out[r] = accumulate ? out[r] + acc : acc;
}

// ---------------------------------------------------------------------------- K7 dedup + top-k
// Each block owns a chunk of entries; k rounds of block argmax by (score desc, order key asc) over
// alive entries, then every alive entry whose schedule equals the winner's is killed (dedup keeps
// the smallest order key, which wins ties).  The order key is the candidate index (final-step
// rounding) or the packed (step, seed) of a history record.  Phase A: entries = candidates, many
// blocks; phase B: entries = phase-A records, one block.  Warp shuffle + shared-memory block reduction.
struct TopkKey { double s; long long o; int c; };
__device__ __forceinline__ bool topk_better(const TopkKey& a, const TopkKey& b) {
  if (a.c < 0) return false;
  if (b.c < 0) return true;
  return a.s > b.s || (a.s == b.s && a.o < b.o);
}
__device__ __forceinline__ TopkKey topk_shfl(const TopkKey& k, int off) {
  return TopkKey{__shfl_xor_sync(0xffffffffu, k.s, off), __shfl_xor_sync(0xffffffffu, k.o, off),
                 __shfl_xor_sync(0xffffffffu, k.c, off)};
}

__global__ void __launch_bounds__(1024) topk_select_kernel(
    long long n_entries, long long chunk, const int* __restrict__ cand_of, const long long* __restrict__ okey,
    const double* __restrict__ score, const unsigned char* __restrict__ valid, const int* __restrict__ sched, int M,
    int k, unsigned char* __restrict__ alive, int* __restrict__ out_cand, int* __restrict__ out_cnt) {
  __shared__ TopkKey red[32];
  __shared__ TopkKey win;
  const long long c0 = static_cast<long long>(blockIdx.x) * chunk;
  const long long c1 = min(n_entries, c0 + chunk);
  for (long long e = c0 + threadIdx.x; e < c1; e += blockDim.x) {
    const int c = cand_of ? cand_of[e] : static_cast<int>(e);
    alive[e] = (c >= 0 && valid[c] && isfinite(score[c])) ? 1 : 0;
  }
  __syncthreads();
  int r = 0;
  for (; r < k; ++r) {
    TopkKey best{0.0, 0, -1};
    for (long long e = c0 + threadIdx.x; e < c1; e += blockDim.x) {
      if (!alive[e]) continue;
      const int c = cand_of ? cand_of[e] : static_cast<int>(e);
      const TopkKey t{score[c], okey ? okey[c] : static_cast<long long>(c), c};
      if (topk_better(t, best)) best = t;
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      const TopkKey o = topk_shfl(best, off);
      if (topk_better(o, best)) best = o;
    }
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = best;
    __syncthreads();
    if (threadIdx.x < 32) {
      TopkKey b = (threadIdx.x < (blockDim.x + 31) / 32) ? red[threadIdx.x] : TopkKey{0.0, 0, -1};
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        const TopkKey o = topk_shfl(b, off);
        if (topk_better(o, b)) b = o;
      }
      if (threadIdx.x == 0) win = b;
    }
    __syncthreads();
    const TopkKey w = win;
    if (w.c < 0) break;
    if (threadIdx.x == 0) out_cand[blockIdx.x * static_cast<long long>(k) + r] = w.c;
    const int* ws = sched + static_cast<size_t>(w.c) * M;
    for (long long e = c0 + threadIdx.x; e < c1; e += blockDim.x) {
      if (!alive[e]) continue;
      const int c = cand_of ? cand_of[e] : static_cast<int>(e);
      const int* cs = sched + static_cast<size_t>(c) * M;
      bool same = true;
      for (int j = 0; j < M; ++j) same = same && (cs[j] == ws[j]);
      if (same) alive[e] = 0;
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    out_cnt[blockIdx.x] = r;
    for (int q = r; q < k; ++q) out_cand[blockIdx.x * static_cast<long long>(k) + q] = -1;
  }
}

// The same selection with the block's entries (score, order key, candidate, alive, schedule) staged in
// shared memory once: the k rounds then touch no global memory (each round of the kernel above pays
// dependent L2 round trips for the scores and the winner's schedule compare).  Identical results.
__global__ void __launch_bounds__(1024) topk_select_smem_kernel(
    long long n_entries, long long chunk, const int* __restrict__ cand_of, const long long* __restrict__ okey,
    const double* __restrict__ score, const unsigned char* __restrict__ valid, const int* __restrict__ sched, int M,
    int k, int* __restrict__ out_cand, int* __restrict__ out_cnt) {
  extern __shared__ double tk_smem[];
  __shared__ TopkKey red[32];
  __shared__ TopkKey win;
  const long long c0 = static_cast<long long>(blockIdx.x) * chunk;
  const int ne = static_cast<int>(min(n_entries, c0 + chunk) - c0);
  double* s_sc = tk_smem;                                            // [chunk]
  long long* s_ok = reinterpret_cast<long long*>(s_sc + chunk);      // [chunk]
  int* s_c = reinterpret_cast<int*>(s_ok + chunk);                   // [chunk]
  int* s_sched = s_c + chunk;                                        // [chunk][M]
  unsigned char* s_alive = reinterpret_cast<unsigned char*>(s_sched + chunk * M);   // [chunk]
  for (int e = threadIdx.x; e < ne; e += blockDim.x) {
    const int c = cand_of ? cand_of[c0 + e] : static_cast<int>(c0 + e);
    const bool live = c >= 0 && valid[c] && isfinite(score[c]);
    s_alive[e] = live ? 1 : 0;
    s_c[e] = c;
    s_sc[e] = live ? score[c] : 0.0;
    s_ok[e] = live ? (okey ? okey[c] : static_cast<long long>(c)) : 0;
    for (int j = 0; j < M; ++j) s_sched[e * M + j] = live ? sched[static_cast<size_t>(c) * M + j] : 0;
  }
  __syncthreads();
  int r = 0;
  for (; r < k; ++r) {
    TopkKey best{0.0, 0, -1};
    int bestE = -1;
    for (int e = threadIdx.x; e < ne; e += blockDim.x) {
      if (!s_alive[e]) continue;
      const TopkKey t{s_sc[e], s_ok[e], s_c[e]};
      if (topk_better(t, best)) { best = t; bestE = e; }
    }
    // carry the entry index in the key's candidate slot's shadow: reduce on (score, order key) as above
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      const TopkKey o = topk_shfl(best, off);
      const int oe = __shfl_xor_sync(0xffffffffu, bestE, off);
      if (topk_better(o, best)) { best = o; bestE = oe; }
    }
    __shared__ int redE[32];
    __shared__ int winE;
    if ((threadIdx.x & 31) == 0) { red[threadIdx.x >> 5] = best; redE[threadIdx.x >> 5] = bestE; }
    __syncthreads();
    if (threadIdx.x < 32) {
      const bool has = threadIdx.x < (blockDim.x + 31) / 32;
      TopkKey b = has ? red[threadIdx.x] : TopkKey{0.0, 0, -1};
      int be = has ? redE[threadIdx.x] : -1;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        const TopkKey o = topk_shfl(b, off);
        const int oe = __shfl_xor_sync(0xffffffffu, be, off);
        if (topk_better(o, b)) { b = o; be = oe; }
      }
      if (threadIdx.x == 0) { win = b; winE = be; }
    }
    __syncthreads();
    const TopkKey w = win;
    if (w.c < 0) break;
    if (threadIdx.x == 0) out_cand[blockIdx.x * static_cast<long long>(k) + r] = w.c;
    const int* ws = s_sched + winE * M;
    for (int e = threadIdx.x; e < ne; e += blockDim.x) {
      if (!s_alive[e]) continue;
      const int* cs = s_sched + e * M;
      bool same = true;
      for (int j = 0; j < M; ++j) same = same && (cs[j] == ws[j]);
      if (same) s_alive[e] = 0;
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    out_cnt[blockIdx.x] = r;
    for (int q = r; q < k; ++q) out_cand[blockIdx.x * static_cast<long long>(k) + q] = -1;
  }
}

// ---------------------------------------------------------------------------- K8 history (Alg. 1 l.13/17/20)
// One thread per seed, run on the rounded point sigma_x_i at which step i's objective is evaluated
// (before the fwd kernel bumps step_ctr to i+1).  A seed whose rounded schedule equals its previous
// step's is skipped; otherwise the schedule is inserted into an open-addressing hash set keyed by the
// full tuple (64-bit hash for the probe, exact tuple compare on a hash match, so distinct schedules are
// never merged).  A new schedule is appended to the pool with key (step << 32 | seed); a repeat lowers
// the stored key with atomicMin, so each pool record ends up with its first (step, seed) occurrence.
__device__ __forceinline__ unsigned long long hist_hash(const int* t, int M) {
  unsigned long long h = 0x9E3779B97F4A7C15ull;
  for (int j = 0; j < M; ++j) {
    h ^= static_cast<unsigned int>(t[j]);
    h *= 0xBF58476D1CE4E5B9ull;
    h ^= h >> 31;
  }
  return h | 1ull;                        // 0 marks an empty slot
}

__global__ void hist_insert_kernel(const int* __restrict__ sched, int n, int M, const int* __restrict__ step_ctr,
                                   int* __restrict__ last, unsigned long long* slot_h, int* slot_i,
                                   unsigned long long slot_mask, int* pool_sched, long long* pool_key, int* pool_cnt,
                                   int pool_cap, int* overflow) {
  const int s = blockIdx.x * blockDim.x + threadIdx.x;
  if (s >= n) return;
  const int step = *step_ctr;
  const int* cur = sched + static_cast<size_t>(s) * M;
  int* lst = last + static_cast<size_t>(s) * M;
  bool changed = (step == 0);
  for (int j = 0; j < M; ++j) changed = changed || (cur[j] != lst[j]);
  if (!changed) return;
  for (int j = 0; j < M; ++j) lst[j] = cur[j];
  const unsigned long long h = hist_hash(cur, M);
  const long long key = (static_cast<long long>(step) << 32) | static_cast<long long>(s);
  unsigned long long p = h & slot_mask;
  for (;;) {
    const unsigned long long prev = atomicCAS(&slot_h[p], 0ull, h);
    if (prev == 0ull) {                                       // claimed: publish a new pool record
      const int idx = atomicAdd(pool_cnt, 1);
      if (idx >= pool_cap) {
        atomicExch(overflow, 1);
        atomicExch(&slot_i[p], -2);
        return;
      }
      for (int j = 0; j < M; ++j) pool_sched[static_cast<size_t>(idx) * M + j] = cur[j];
      pool_key[idx] = key;
      __threadfence();
      atomicExch(&slot_i[p], idx);
      return;
    }
    if (prev == h) {                                          // same hash: wait for the record, compare
      int idx;
      while ((idx = atomicAdd(&slot_i[p], 0)) == -1) {}
      if (idx == -2) return;
      __threadfence();
      const int* ps = pool_sched + static_cast<size_t>(idx) * M;
      bool same = true;
      for (int j = 0; j < M; ++j) same = same && (ps[j] == cur[j]);
      if (same) {
        atomicMin(&pool_key[idx], key);
        return;
      }
    }
    p = (p + 1) & slot_mask;
  }
}

// history records -> host arrays: global index = index_base + seed, step
__global__ void hist_gather_kernel(const int* __restrict__ cand, const int* __restrict__ cnt, int k,
                                   const double* __restrict__ score, const int* __restrict__ sched,
                                   const long long* __restrict__ key, int M, long long index_base,
                                   long long* __restrict__ o_idx, int* __restrict__ o_step, double* __restrict__ o_score,
                                   int* __restrict__ o_sched) {
  const int r = threadIdx.x;
  if (r >= k) return;
  const int c = r < cnt[0] ? cand[r] : -1;
  o_idx[r] = c >= 0 ? index_base + (key[c] & 0xffffffffll) : -1;
  o_step[r] = c >= 0 ? static_cast<int>(key[c] >> 32) : -1;
  o_score[r] = c >= 0 ? score[c] : 0.0;
  for (int j = 0; j < M; ++j) o_sched[static_cast<size_t>(r) * M + j] = c >= 0 ? sched[static_cast<size_t>(c) * M + j] : 0;
}

// gather the final records into contiguous arrays for one D2H copy
__global__ void topk_gather_kernel(const int* __restrict__ cand, const int* __restrict__ cnt, int k, const double* __restrict__ score,
                                   const int* __restrict__ sched, int M, long long index_base,
                                   long long* __restrict__ o_idx, double* __restrict__ o_score, int* __restrict__ o_sched) {
  const int r = threadIdx.x;
  if (r >= k) return;
  const int c = r < cnt[0] ? cand[r] : -1;
  o_idx[r] = c >= 0 ? index_base + c : -1;
  o_score[r] = c >= 0 ? score[c] : 0.0;
  for (int j = 0; j < M; ++j) o_sched[static_cast<size_t>(r) * M + j] = c >= 0 ? sched[static_cast<size_t>(c) * M + j] : 0;
}

}  // namespace felix
