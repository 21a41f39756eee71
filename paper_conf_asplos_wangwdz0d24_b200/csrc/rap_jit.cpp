// rap_jit.cpp — plan-specialised row-block kernel: a code generator plus
// NVRTC (the B200-native form of RAP's code generator, §4
// L854-857: the optimizer's plan becomes "optimized CUDA kernels").
//
// For a plan, the generator writes one policy for the row-block kernel
// skeleton (rap_rows_skel.cuh): every sparse output's closed-form length and
// its chain as straight-line code, in the planner's processing order, with
// every parameter (caps, fills, Clamp bounds, H(salt), M, MapId / Bucketize
// table offsets) an immediate and the staged column slots constants.  An
// NGram output over sources another output already hashed reads them from
// registers (the provider's element 0, rows with at most one id).  Anything
// else (non-canonical chains, dense-bucket sources, rows with longer lists)
// calls the interpreter's generic functions (rap_rows_interp.cuh), so the
// generated kernel computes exactly what the interpreter computes (R1-R20).
// The source is compiled with NVRTC for sm_100a once per distinct plan source
// in the process and loaded as a cudaLibrary; the launch path is the same
// cooperative launch as rap_rows.cu.
#include <cuda_runtime.h>
#include <nvrtc.h>
#include <math.h>
#include <stdio.h>
#include <string.h>

#include <algorithm>
#include <chrono>
#include <cstdlib>
#include <cinttypes>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "rap_internal.h"

namespace rapk {

// Header texts (generated from the csrc/ headers at build time by _build.py).
#include "rap_jit_embed.inc"

static int env_int(const char* name, int dflt) {
  const char* e = getenv(name);
  return (e && *e) ? atoi(e) : dflt;
}

struct JitModule {
  cudaLibrary_t lib = nullptr;
  cudaKernel_t k = nullptr;
  double compile_s = 0;
};

namespace {

std::string lit64(int64_t v) {
  if (v == INT64_MIN) return "(-9223372036854775807LL - 1LL)";
  return std::to_string(v) + "LL";
}
std::string litu64(uint64_t v) { return std::to_string(v) + "ULL"; }
std::string i2s(long long v) { return std::to_string(v); }
std::string f2lit(float f) {  // exact (hex float)
  if (f != f) return "__int_as_float(0x7fc00000)";
  if (f == INFINITY) return "__int_as_float(0x7f800000)";
  if (f == -INFINITY) return "__int_as_float(0xff800000)";
  char buf[64];
  snprintf(buf, sizeof(buf), "%af", (double)f);
  return buf;
}

struct Gen {
  const JitPlanView& v;
  int F;
  std::vector<int> slot;     // raw column -> staged slot (rank among the columns the outputs read)
  std::vector<int> provider; // per output f: a memo provider for NGram source i? see prov_out
  std::string out;

  explicit Gen(const JitPlanView& view) : v(view), F(view.n_sparse_out) {
    std::vector<char> used(std::max(1, view.n_sparse_in), 0);
    for (int f = 0; f < F; ++f) {
      const RbFeat& R = v.feat[f];
      const int kk = R.kind == 1 ? 0 : R.k;
      for (int i = 0; i < kk; ++i)
        if (R.src[i] >= 0) used[R.src[i]] = 1;
    }
    slot.assign(used.size(), -1);
    int n = 0;
    for (size_t c = 0; c < used.size(); ++c)
      if (used[c]) slot[c] = n++;
    plan_tables();
  }

  // ---- Bucketize tables staged in shared memory at launch ----
  // The three-level search's two bursts (8 sub-block maxima, then 8 borders)
  // are dependent L2 round trips on every row's chain; with the tables in
  // shared memory they are two shared loads.  Sample tables of every 3-level
  // Bucketize first (1 KB per 1024 borders), then whole border tables while
  // the budget lasts (the rest keep their borders in global).
  struct BkTab {
    int64_t a;
    int m;
    int off_s, off_b;  // byte offsets after the 16-byte mbarrier (off_b < 0: borders in global)
  };
  std::vector<BkTab> bktabs;
  int tab_total = 0;  // bytes after the mbarrier
  // 8 KB: the sample tables (whole border tables would cost C2 its second
  // CTA per SM: measured 41 -> 65 us with 36 KB of tables)
  static int tab_budget() { return env_int("RAP_JIT_TABS", 1) ? env_int("RAP_JIT_TAB_BYTES", 8 * 1024) : 0; }
  void plan_tables() {
    std::vector<std::pair<int64_t, int>> want;
    for (int f = 0; f < F; ++f) {
      if (v.feat[f].emit != 0 && v.feat[f].emit != 3) continue;
      const Canon& q = v.sprogs[f].cn;
      if (!(q.mask & CB_BUCKET)) continue;
      if (!(q.bk_m >= 64 && q.bk_m % 64 == 0 && q.bk_a % 2 == 0)) continue;
      bool seen = false;
      for (const auto& w : want) seen |= w.first == q.bk_a;
      if (!seen) want.push_back({q.bk_a, q.bk_m});
    }
    const int budget = tab_budget();
    for (const auto& w : want) {
      const int sb = (w.second / 8) * 8;
      if (tab_total + sb > budget) break;
      bktabs.push_back(BkTab{w.first, w.second, tab_total, -1});
      tab_total += sb;
    }
    for (BkTab& t : bktabs) {
      const int bb = t.m * 8;
      if (tab_total + bb > budget) continue;
      t.off_b = tab_total;
      tab_total += bb;
    }
  }
  const BkTab* staged_table(int64_t a) const {
    for (const BkTab& t : bktabs)
      if (t.a == a) return &t;
    return nullptr;
  }
  int table_bytes() const { return tab_total > 0 ? 16 + tab_total : 0; }
  std::string setup_tables() {
    if (tab_total == 0) return "";
    std::string s = "    if (threadIdx.x == 0 && x.FL > 0 && x.R1 > x.R0) {  // the plan's tables -> shared memory\n"
                    "      uint64_t* bar = reinterpret_cast<uint64_t*>(s.tabs);\n"
                    "      mbar_init(bar, 1);\n"
                    "      mbar_arrive_expect(bar, " + i2s(tab_total) + "u);\n";
    for (const BkTab& t : bktabs) {
      s += "      bulk_g2s(s.tabs + " + i2s(16 + t.off_s) + ", " + sample_table(t.a, t.m) + ", " + i2s((t.m / 8) * 8) +
           "u, bar);\n";
      if (t.off_b >= 0)
        s += "      bulk_g2s(s.tabs + " + i2s(16 + t.off_b) + ", p.c.itab + " + lit64(t.a) + ", " + i2s(t.m * 8) + "u, bar);\n";
    }
    return s + "    }\n";
  }

  static std::string cap_expr(const std::string& X, int cap) {
    if (cap >= INT32_MAX) return "max(" + X + ".b - " + X + ".a, 0)";
    return "min(max(" + X + ".b - " + X + ".a, 0), " + i2s(cap) + ")";
  }

  // int32_t L<q> (and RbRow X<q>_<i>, int32_t l<q>_<i> for NGram sources)
  std::string len_code(int q) {
    const int f = v.perm[q];
    const RbFeat& R = v.feat[f];
    const std::string Q = i2s(q);
    std::string s;
    if (R.kind == 1) return "    const int32_t L" + Q + " = in ? " + i2s(R.out_cap) + " : 0;\n";
    if (R.kind == 0) {
      const std::string X = "X" + Q + "_0";
      s += "    const RbRow " + X + " = " + rbrow() + "(s, " + i2s(slot[R.src[0]]) + ", r);\n";
      s += "    const int32_t L" + Q + " = in ? (" + X + ".valid ? " + cap_expr(X, R.cap[0]) + " : " + i2s(R.ncap[0]) +
           ") : 0;\n";
      return s;
    }
    std::string sum = "0LL";
    for (int i = 0; i < R.k; ++i) {
      const std::string l = "l" + Q + "_" + i2s(i);
      if (R.src[i] < 0) {
        s += "    const int32_t " + l + " = " + i2s(R.cap[i]) + ";\n";
      } else {
        const std::string X = "X" + Q + "_" + i2s(i);
        s += "    const RbRow " + X + " = " + rbrow() + "(s, " + i2s(slot[R.src[i]]) + ", r);\n";
        s += "    const int32_t " + l + " = " + X + ".valid ? " + cap_expr(X, R.cap[i]) + " : " + i2s(R.ncap[i]) +
             ";\n";
      }
      sum += " + " + l;
    }
    s += "    const int32_t L" + Q + " = in ? (int32_t)min(max((long long)(" + sum + ") - " + i2s(R.n) +
         "LL + 1LL, 0LL), " + i2s(R.out_cap) + "LL) : 0;\n";
    return s;
  }

  // Canonical stages (R6, R8, R1-R3, R4) on variable x; memo: store after
  // stage bit memo_after into variable mvar (16: before the first stage).
  std::string stages(const Canon& q, int mask, const std::string& x, const std::string& full, int memo_after,
                     const std::string& mvar, const std::string& probe = "") {
    std::string s;
    // (experiment knob RAP_JIT_SKIP: bit 1 MapId, 2 SigridHash, 4 Bucketize
    // stages left out -- wrong outputs, for cost attribution only)
    mask &= ~(env_int("RAP_JIT_SKIP", 0) & 1 ? CB_MAPID : 0);
    mask &= ~(env_int("RAP_JIT_SKIP", 0) & 2 ? CB_SIGRID : 0);
    mask &= ~(env_int("RAP_JIT_SKIP", 0) & 4 ? CB_BUCKET : 0);
    auto cond = [&](int bit) { return (q.null_mask & bit) ? std::string() : "if (" + full + ") "; };
    if (memo_after == 16) s += "        " + mvar + " = " + x + ";\n";
    if (mask & CB_CLAMP) {
      s += "        " + cond(CB_CLAMP) + "{ " + x + " = " + x + " < " + lit64(q.lo) + " ? " + lit64(q.lo) + " : " + x +
           "; " + x + " = " + x + " > " + lit64(q.hi) + " ? " + lit64(q.hi) + " : " + x + "; }\n";
      if (memo_after == CB_CLAMP) s += "        " + mvar + " = " + x + ";\n";
    }
    if (mask & CB_MAPID) {
      if (!probe.empty())  // first probe loaded ahead
        s += "        " + cond(CB_MAPID) + x + " = " + (map2() ? "map_lookup_from2" : "map_lookup_from") + "(c.itab, " + lit64(q.map_a) + ", " + i2s(q.map_m) + ", " +
             lit64(q.map_def) + ", " + x + ", " + probe + ");\n";
      else
        s += "        " + cond(CB_MAPID) + x + " = map_lookup(c.itab, " + lit64(q.map_a) + ", " + i2s(q.map_m) + ", " +
             lit64(q.map_def) + ", 0, 0, " + x + ");\n";
      if (memo_after == CB_MAPID) s += "        " + mvar + " = " + x + ";\n";
    }
    if (mask & CB_SIGRID) {
      s += "        " + cond(CB_SIGRID) + x + " = (int64_t)reduce_M(splitmix_H(" + litu64(q.hs) + " ^ (uint64_t)" + x +
           "), " + lit64(q.M) + ");\n";
      if (memo_after == CB_SIGRID) s += "        " + mvar + " = " + x + ";\n";
    }
    if (mask & CB_BUCKET) {
      if (q.bk_m >= 64 && q.bk_m % 64 == 0 && q.bk_a % 2 == 0) {
        // three levels: the maxima of the 64-border blocks as immediates, then
        // one burst of 8 sub-block maxima and one of 8 borders (R4)
        const std::string nm = sample_table(q.bk_a, q.bk_m);
        s += "        " + cond(CB_BUCKET) + "{ const int j0 = 0";
        for (int k = 0; k < q.bk_m / 64; ++k) s += " + (" + x + " >= " + lit64(v.itab[q.bk_a + 64 * k + 63]) + ")";
        const BkTab* t = staged_table(q.bk_a);
        const std::string smp =
            t ? "reinterpret_cast<const int64_t*>(s.tabs + " + i2s(16 + t->off_s) + ")" : nm;
        const std::string brd = (t && t->off_b >= 0)
                                    ? "reinterpret_cast<const int64_t*>(s.tabs + " + i2s(16 + t->off_b) + ")"
                                    : "c.itab + " + lit64(q.bk_a);
        const std::string fn = !t ? "upper_bound_64" : (t->off_b >= 0 ? "upper_bound_64s" : "upper_bound_64h");
        s += "; " + x + " = " + fn + "(" + brd + ", " + i2s(q.bk_m) + ", " + smp + ", j0, " + x + "); }\n";
      } else if (q.bk_m >= 64) {  // two-level search over a sample table in the module
        const std::string nm = sample_table(q.bk_a, q.bk_m);
        s += "        " + cond(CB_BUCKET) + x + " = upper_bound_s8(c.itab + " + lit64(q.bk_a) + ", " + i2s(q.bk_m) +
             ", " + nm + ", " + i2s(q.bk_m / 8) + ", " + x + ");\n";
      } else {
        s += "        " + cond(CB_BUCKET) + x + " = upper_bound(c.itab + " + lit64(q.bk_a) + ", " + i2s(q.bk_m) + ", " +
             x + ");\n";
      }
      if (memo_after == CB_BUCKET) s += "        " + mvar + " = " + x + ";\n";
    }
    return s;
  }

  // __device__ table of every 8th border of itab[a .. a+m) (upper_bound_s8)
  std::map<int64_t, std::string> samples;
  std::string sample_globals;
  std::string sample_table(int64_t a, int m) {
    auto it = samples.find(a);
    if (it != samples.end()) return it->second;
    const std::string nm = "kS" + i2s((long long)samples.size());
    sample_globals += "__device__ __align__(16) const int64_t " + nm + "[" + i2s(std::max(1, m / 8)) + "] = {";
    for (int i = 0; i < m / 8; ++i) sample_globals += (i ? ", " : "") + lit64(v.itab[a + 8 * i + 7]);
    if (m / 8 == 0) sample_globals += "0";
    sample_globals += "};\n";
    samples[a] = nm;
    return nm;
  }

  // upper bound of an output's row length (its FirstX caps), for the scans
  int max_len(int f) const {
    const RbFeat& R = v.feat[f];
    if (R.kind == 1) return R.out_cap;
    if (R.kind == 0) return std::max(R.cap[0], R.ncap[0]);
    long long t = 0;
    for (int i = 0; i < R.k; ++i) t += std::max(R.cap[i], R.ncap[i]);
    return (int)std::min<long long>(std::max(0LL, t - R.n + 1), R.out_cap);
  }

  static int memo_point(const RbFeat& R, const Canon& cn) {
    if (R.memo_slot < 0) return -1;
    const int pm = R.memo_mask & cn.mask;
    if (pm == 0) return 16;
    int ma = 1;
    while ((pm >> 1) >= ma) ma <<= 1;
    return ma;
  }

  // ---- dense outputs (a2): thread per row, units split over two halves ----
  int pitch() const { return v.d_out | 1; }
  // the dense warp's tile sits after the base-phase totals T[f], L[f]
  int tile_offset() const { return ((2 * (F + 1) * 8) + 15) & ~15; }
  int dense_mode() const {
    int r0 = 0;
    return jit_dense_mode(F, v.d_out, v.n_dprogs, v.dense_bytes, v.pairs, &r0);
  }
  bool gen_dense_ok() const { return dense_mode() == 1 || dense_mode() == 3; }  // the dense-warp forms (kDenseWarp)
  int threads() const {
    if (pairs()) return 2 * kRbChunk;
    const int nd = jit_dense_warps(dense_mode());
    return nd ? 224 + 32 * nd : kRbChunk;
  }
  double unit_cost(const DProg& dp, const DUnit& un) const {
    const DevOp* ops = un.gops ? v.ops : dp.ops;
    double c = 8;
    if (un.kind == U_ONEHOT_G) return 200;
    for (int o = un.op_begin; o < un.op_end; ++o)
        c += ops[o].kind == OK_LOGIT ? 40 : ops[o].kind == OK_BOXCOX ? 70 : 3;
    if (un.kind == U_ONEHOT_DB) c += 10 + un.width + un.bm / 2;
    return c;
  }
  std::string dense_ops(const DevOp* ops, int o0, int o1, const std::string& x) {
    std::string s;
    for (int o = o0; o < o1; ++o) {
      const DevOp& op = ops[o];
      if (op.kind == OK_FILL_F) {
        s += "        if (isnan(" + x + ")) " + x + " = " + f2lit(op.f0) + ";\n";  // R10
      } else if (op.kind == OK_LOGIT) {                                          // R11
        s += "        { const float z = " + x + " < " + f2lit(op.f0) + " ? " + f2lit(op.f0) + " : (" + x + " > " +
             f2lit(op.f1) + " ? " + f2lit(op.f1) + " : " + x + "); " + x + " = logf(__fdiv_rn(z, __fsub_rn(1.0f, z))); }\n";
      } else if (op.f0 == 0.0f) {  // R12, lambda = 0
        s += "        " + x + " = logf(" + x + ");\n";
      } else {  // R12
        s += "        " + x + " = __fdiv_rn(expm1f(__fmul_rn(" + f2lit(op.f0) + ", logf(" + x + "))), " + f2lit(op.f0) +
             ");\n";
      }
    }
    return s;
  }
  std::string id_ops(const DevOp* ops, int o0, int o1, const std::string& b) {
    std::string s;
    for (int o = o0; o < o1; ++o) {
      const DevOp& op = ops[o];
      if (op.kind == OK_CLAMP) {
        s += "        " + b + " = " + b + " < " + lit64(op.a) + " ? " + lit64(op.a) + " : " + b + "; " + b + " = " + b +
             " > " + lit64(op.b) + " ? " + lit64(op.b) + " : " + b + ";\n";
      } else if (op.kind == OK_SIGRID) {
        s += "        " + b + " = (int64_t)reduce_M(splitmix_H(" + litu64(op.hsalt) + " ^ (uint64_t)" + b + "), " +
             lit64(op.M) + ");\n";
      } else if (op.kind == OK_BUCKET_I) {
        s += "        " + b + " = upper_bound(c.itab + " + lit64(op.a) + ", " + i2s(op.m) + ", " + b + ");\n";
      } else {  // OK_MAPID
        s += "        " + b + " = map_lookup(c.itab, " + lit64(op.a) + ", " + i2s(op.m) + ", " + lit64(op.b) + ", " +
             i2s((int)op.M) + ", " + lit64((int64_t)op.hsalt) + ", " + b + ");\n";
      }
    }
    return s;
  }
  std::string dense_unit(int gi, int ui, std::string* globals) {
    const DProg& dp = v.dprogs[gi];
    const DUnit& un = dp.units[ui];
    const int col = dp.col0 + un.col;  // absolute output column
    std::string s = "      {  // dense unit " + i2s(gi) + "." + i2s(ui) + "\n";
    if (un.kind == U_ONEHOT_G) {  // generic list (R9): the interpreter's code
      s += "        for (int k = 0; k < " + i2s(un.width) + "; ++k) trow[" + i2s(col) + " + k] = 0.0f;\n";
      s += "        onehot_generic(p, p.c.dprogs[" + i2s(gi) + "].units[" + i2s(ui) + "], row, trow + " + i2s(dp.col0) +
           ");\n      }\n";
      return s;
    }
    s += "        float v = in" + i2s(un.src_col) + ";\n";
    const DevOp* uops = un.gops ? v.ops : dp.ops;  // gops: indices into the global pools
    s += dense_ops(uops, un.op_begin, un.op_end, "v");
    if (un.kind == U_DENSE) {
      s += "        trow[" + i2s(col) + "] = v;\n      }\n";
      return s;
    }
    // U_ONEHOT_DB: Bucketize (f32 borders, R4) -> id ops -> OneHot (R9)
    if (un.xcap <= 0) {
      s += "        for (int k = 0; k < " + i2s(un.width) + "; ++k) trow[" + i2s(col) + " + k] = 0.0f;\n      }\n";
      return s;
    }
    const float* bt = (un.gops ? v.ftab : dp.ftab) + un.btab;
    if (un.bm <= 32) {
      s += "        int64_t b = 0";
      for (int i = 0; i < un.bm; ++i) s += " + (v >= " + f2lit(bt[i]) + ")";
      s += ";\n";
    } else {
      const std::string nm = "kB" + i2s(gi) + "_" + i2s(ui);
      *globals += "__device__ const float " + nm + "[" + i2s(un.bm) + "] = {";
      for (int i = 0; i < un.bm; ++i) *globals += (i ? ", " : "") + f2lit(bt[i]);
      *globals += "};\n";
      s += "        int64_t b = upper_bound(" + nm + ", " + i2s(un.bm) + ", v);\n";
    }
    s += id_ops(uops, un.iop_begin, un.iop_end, "b");
    s += "        const int64_t d = b - " + lit64(un.k0) + ";\n";
    s += "#pragma unroll\n        for (int k = 0; k < " + i2s(un.width) + "; ++k) trow[" + i2s(col) +
         " + k] = d == k ? 1.0f : 0.0f;\n      }\n";
    return s;
  }
  std::string dense_fn(std::string* globals) {
    // the dense warp (warp 7): its lane = a row of the block, every unit of
    // the row (independent loads first), a 32-row tile in shared memory after
    // the base-phase totals, then stored by the warp
    std::string s;
    const int mode = dense_mode();
    const bool ok = mode == 1 || mode == 3;
    s += "  static constexpr bool kGenDense = " + std::string(mode == 2 ? "true" : "false") + ";\n";
    s += "  static constexpr bool kDenseWarp = " + std::string(ok ? "true" : "false") + ";\n";
    if (mode == 2) {
      s += "  template <class P>\n  static __device__ __forceinline__ void dense_warp(const P&, const RbSmem&, const RbCtx&) {}\n";
      s += "  template <class P>\n  static __device__ __forceinline__ void dense(const P& p, const RbSmem& s, const RbCtx& x) {\n";
    } else {
      s += "  template <class P>\n  static __device__ __forceinline__ void dense(const P&, const RbSmem&, const RbCtx&) {}\n";
      s += "  template <class P>\n  static __device__ __forceinline__ void dense_warp(const P& p, const RbSmem& s, const RbCtx& x) {\n";
      if (!ok) return s + "  }\n";
    }
    std::vector<std::pair<int, int>> units;
    std::vector<int> cols;
    for (int gi = 0; gi < v.n_dprogs; ++gi)
      for (int ui = 0; ui < v.dprogs[gi].n_units; ++ui) {
        units.push_back({gi, ui});
        const DUnit& un = v.dprogs[gi].units[ui];
        if (un.kind != U_ONEHOT_G && std::find(cols.begin(), cols.end(), un.src_col) == cols.end())
          cols.push_back(un.src_col);
      }
    s += "    const Common& c = p.c;\n    const int lane = threadIdx.x & 31;\n";
    if (mode == 2) {  // warps < nt: their own tile, 32-row tiles of the block round robin over them
      const int nt = jit_dense_tiles(v.pairs);
      s += "    const int warp = threadIdx.x >> 5;\n";
      s += "    float* tile = reinterpret_cast<float*>(s.dense + " + i2s(tile_offset()) + ") + warp * " +
           i2s(32 * pitch()) + ";  // [" + i2s(nt) + "][32][" + i2s(pitch()) + "]\n";
      s += "    if (warp < " + i2s(nt) + ")\n";
      s += "    for (int64_t d0 = x.R0 + 32 * warp; d0 < x.R1; d0 += " + i2s(32 * nt) + ") {\n";
    } else {  // dense warps 7 .. 7 + nd - 1: their own tile, the block's 32-row tiles round robin over them
      const int nd = jit_dense_warps(mode);
      s += "    const int dw = (threadIdx.x >> 5) - 7;\n";
      s += "    float* tile = reinterpret_cast<float*>(s.dense + " + i2s(tile_offset()) + ") + dw * " + i2s(32 * pitch()) +
           ";  // [" + i2s(nd) + "][32][" + i2s(pitch()) + "]\n";
      s += "    for (int64_t d0 = x.R0 + 32 * dw; d0 < x.R1; d0 += " + i2s(32 * nd) + ") {\n";
    }
    s += "      const int nr = (int)min((int64_t)32, x.R1 - d0);\n";
    s += "      if (lane < nr) {\n        const int64_t row = d0 + lane;\n";
    s += "        float* trow = tile + lane * " + i2s(pitch()) + ";\n";
    for (int cc : cols) s += "        const float in" + i2s(cc) + " = rb_dense_in(p, " + i2s(cc) + ", row);\n";
    for (const auto& u : units) s += dense_unit(u.first, u.second, globals);
    s += "      }\n      __syncwarp();\n";
    s += "      rb_tile_store_warp(c, tile, " + i2s(pitch()) + ", " + i2s(v.d_out) + ", d0, nr);\n      __syncwarp();\n    }\n  }\n";
    return s;
  }

  // Warp-pair mode (rap_rows_skel.cuh kPairs): warps 2w, 2w + 1 take the
  // outputs [0, split) and [split, F) of the processing order over the same
  // 32 rows.  split: a unit boundary (no NGram separated from a memo provider)
  // nearest to half the predicted cost.
  bool pairs() const { return v.pairs != 0; }
  // programmatic dependent launch of consecutive launches (experiment knob)
  static bool jit_pdl() { return env_int("RAP_JIT_PDL", 0) != 0; }
  // MapId: the first two probe slots loaded ahead (RAP_JIT_MAP1=1: one, experiment knob)
  static bool map2() { return env_int("RAP_JIT_MAP1", 0) == 0; }
  std::string rbrow() const { return "rb_row_p<" + i2s(kRbChunk + 4) + ">"; }
  std::string thread_vars() const {
    if (pairs())
      return "    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, wi = warp >> 1, r = (wi << 5) | lane;\n"
             "    (void)tid;\n";
    return "    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, wi = warp, r = tid;\n"
           "    (void)lane;\n    (void)wi;\n";
  }
  int split_point() const {
    if (!pairs()) return F;
    double tot = 0;
    std::vector<double> pre(F + 1, 0.0);
    for (int q = 0; q < F; ++q) pre[q + 1] = pre[q] + out_cost(q);
    tot = pre[F];
    int best = F;
    double bd = 1e30;
    for (int sp = 1; sp < F; ++sp) {
      bool ok = true;  // no NGram at >= sp reads a memo provider at < sp
      for (int q = sp; q < F && ok; ++q) {
        const RbFeat& R = v.feat[v.perm[q]];
        if (R.emit != 3) continue;
        for (int i = 0; i < R.k; ++i)
          if (R.prov[i] >= 0 && R.prov[i] < sp) ok = false;
      }
      if (!ok) continue;
      const double d = std::fabs(pre[sp] - 0.5 * tot);
      if (d < bd) {
        bd = d;
        best = sp;
      }
    }
    return best;
  }
  std::string lengths_fn() {
    std::string s;
    s += "  template <bool kSmall, class P>\n"
         "  static __device__ __forceinline__ void lengths(const P& p, const RbSmem& s, const RbCtx& x, int nr, "
         "bool acc) {\n" + thread_vars() +
         "    const bool in = r < nr;\n";
    const int sp = split_point();
    if (pairs()) s += "  if ((warp & 1) == 0) {\n";
    s += lengths_body(0, sp);
    if (pairs()) s += "  } else {\n" + lengths_body(sp, F) + "  }\n";
    s += "  }\n";
    return s;
  }
  std::string lengths_body(int qb, int qe) {
    std::string s;
    // batches of 8 outputs: every staged load of a batch before its warp sums
    // are stored (a shared store would otherwise order the next loads)
    for (int q0 = qb; q0 < qe; q0 += 8) {
      const int q1 = std::min(qe, q0 + 8);
      s += "  {\n";
      for (int q = q0; q < q1; ++q) s += len_code(q);
      for (int q = q0; q < q1; ++q) s += "    const long long w" + i2s(q) + " = rb_warp_sum<kSmall>(L" + i2s(q) + ");\n";
      s += "    if (lane == 0) {\n";
      for (int q = q0; q < q1; ++q)
        s += "      s.ws[" + i2s(q * 8) + " + wi] = acc ? s.ws[" + i2s(q * 8) + " + wi] + w" + i2s(q) + " : w" + i2s(q) +
             ";\n";
      s += "    }\n  }\n";
    }
    return s;
  }

  // ---- dense-warp tail: the last outputs of the processing order (whole
  // NGram units, ~tail_frac of the predicted cost) are emitted by the dense
  // warps once their tiles are done, one row warp at a time, so the sparse
  // warps' chains are that much shorter (one-chunk blocks, dense mode 3) ----
  int tail_split() const {
    if (!batch_ok() || pairs() || dense_mode() != 3 || loop_plan_ok()) return F;
    const double frac = env_int("RAP_JIT_TAIL_PCT", 20) / 100.0;
    if (frac <= 0) return F;
    std::vector<double> pre(F + 1, 0.0);
    for (int q = 0; q < F; ++q) pre[q + 1] = pre[q] + out_cost(q);
    int best = F;
    double bd = 1e30;
    for (int sp = std::min(F, batch_k()); sp < F; ++sp) {  // the tail never takes batch 0 (pre_emit)
      bool ok = true;
      for (int q = sp; q < F && ok; ++q) {
        const RbFeat& R = v.feat[v.perm[q]];
        if (R.emit != 3) continue;
        for (int i = 0; i < R.k; ++i)
          if (R.prov[i] >= 0 && R.prov[i] < sp) ok = false;
      }
      if (!ok) continue;
      const double d = std::fabs((pre[F] - pre[sp]) - frac * pre[F]);
      if (d < bd) {
        bd = d;
        best = sp;
      }
    }
    return best;
  }
  bool loop_plan_ok() const { return const_cast<Gen*>(this)->loop_plan().ok; }
  std::string emit_fn() {
    std::string s;
    s += "  template <bool kSmall, class P>\n"
         "  static __device__ __forceinline__ void emit(const P& p, const RbSmem& s, const RbCtx& x, int64_t c0, "
         "int nr, const PreState& ps, bool use_pre, bool tail_by_dense) {\n" + thread_vars() +
         "    const Common& c = p.c;\n"
         "    const int64_t B = x.B;\n"
         "    const bool in = r < nr;\n"
         "    const int64_t row = c0 + r;\n    (void)ps;\n    (void)use_pre;\n    (void)tail_by_dense;\n";
    const int sp = split_point();
    if (tab_total) s += "    mbar_wait(reinterpret_cast<uint64_t*>(s.tabs), 0u);  // staged tables landed\n";
    const LoopPlan lp = loop_plan();
    if (lp.ok) return s + emit_loop(lp) + "  }\n" + tail_fn(F);
    if (pairs()) s += "  if ((warp & 1) == 0) {\n";
    const int ts = pairs() ? F : tail_split();
    if (batch_ok() && ts < F) {
      s += "  {\n" + emit_batched(0, ts) + "  }\n";
      s += "  if (!tail_by_dense) {\n" + emit_batched(ts, F) + "  }\n";
    } else {
      s += batch_ok() ? emit_batched(0, sp) : emit_body(0, sp);
    }
    if (pairs()) s += "  } else {\n" + (batch_ok() ? emit_batched(sp, F) : emit_body(sp, F)) + "  }\n";
    s += "  }\n";
    return s + tail_fn(ts);
  }
  // emit_tail: the outputs [ts, F) of row warp w of the chunk, by a dense warp
  std::string tail_fn(int ts) {
    std::string s = "  static constexpr bool kTail = " + std::string(ts < F ? "true" : "false") + ";\n";
    s += "  template <bool kSmall, class P>\n"
         "  static __device__ __forceinline__ void emit_tail(const P& p, const RbSmem& s, const RbCtx& x, int64_t c0, "
         "int nr, int w) {\n";
    if (ts >= F) return s + "  }\n";
    s += "    const int lane = threadIdx.x & 31, wi = w, r = (w << 5) | lane;\n"
         "    const Common& c = p.c;\n"
         "    const int64_t B = x.B;\n"
         "    const bool in = r < nr;\n"
         "    const int64_t row = c0 + r;\n"
         "    const bool use_pre = false;\n    (void)use_pre;\n";
    if (tab_total) s += "    mbar_wait(reinterpret_cast<uint64_t*>(s.tabs), 0u);\n";
    s += emit_batched(ts, F);
    return s + "  }\n";
  }
  // ---- loop emitter (rap_rows_skel.cuh jl_*): the outputs as rows of
  // __constant__ tables, NGram units (k providers + the NGram) then single
  // canonical outputs in two loops, so the code a warp streams through in the
  // emit phase is two short loop bodies (ncu: instruction-fetch stalls were
  // 40% of the straight-line emitters' warp samples) ----
  struct LoopPlan {
    bool ok = false;
    int K = 0, N = 0;
    std::vector<int> canon;  // processing indices: unit u's providers at [u*K, u*K+K), then the singles
    std::vector<int> units;  // processing index of each unit's NGram
    std::vector<int64_t> bk; // distinct Bucketize border offsets (rows of the level-0 / sample tables)
  };
  LoopPlan loop_plan() {
    LoopPlan L;
    // opt-in (RAP_JIT_LOOP=1): measured on C2, the loops' serial chains cost
    // more than the instruction fetches they save (emit phase 19 -> 28 us)
    if (env_int("RAP_JIT_LOOP", 0) == 0 || pairs() || column_mode()) return L;
    std::vector<char> used(F, 0);
    for (int q = 0; q < F; ++q) {
      const int f = v.perm[q];
      const RbFeat& R = v.feat[f];
      const SProg& pg = v.sprogs[f];
      if (R.emit == 0) {
        const Canon& cn = pg.cn;
        if (!cn.ok || R.kind != 0 || max_len(f) > 1) return L;
        if (cn.mask & CB_BUCKET) {
          if (!(cn.bk_m >= 64 && cn.bk_m <= 1024 && cn.bk_m % 64 == 0 && cn.bk_a % 2 == 0)) return L;
          if (std::find(L.bk.begin(), L.bk.end(), cn.bk_a) == L.bk.end()) L.bk.push_back(cn.bk_a);
        }
      } else if (R.emit == 3) {
        if (!ngram_fast_ok(q) || pg.cn.mask != 0 || R.k > kMaxNgramK || R.n > R.k) return L;
        if (L.K == 0) {
          L.K = R.k;
          L.N = R.n;
        }
        if (R.k != L.K || R.n != L.N) return L;
        for (int i = 0; i < R.k; ++i)
          if (R.prov[i] != q - R.k + i || used[q - R.k + i]) return L;
        for (int i = 0; i < R.k; ++i) used[q - R.k + i] = 1;
        L.units.push_back(q);
      } else {
        return L;
      }
    }
    if ((int)L.units.size() > 32) return L;
    for (int u : L.units)
      for (int i = 0; i < L.K; ++i) L.canon.push_back(u - L.K + i);
    for (int q = 0; q < F; ++q)
      if (v.feat[v.perm[q]].emit == 0 && !used[q]) L.canon.push_back(q);
    L.ok = true;
    return L;
  }
  std::string loop_tables(const LoopPlan& L) {
    std::string s;
    s += "__constant__ rapk::JLCanon kJC[" + i2s(std::max<size_t>(1, L.canon.size())) + "] = {\n";
    for (int q : L.canon) {
      const int f = v.perm[q];
      const RbFeat& R = v.feat[f];
      const SProg& pg = v.sprogs[f];
      const Canon& cn = pg.cn;
      int bk_row = 0;
      if (cn.mask & CB_BUCKET) bk_row = (int)(std::find(L.bk.begin(), L.bk.end(), cn.bk_a) - L.bk.begin());
      const int mp = R.memo_slot >= 0 ? memo_point(R, cn) : -1;
      s += "  {" + lit64(pg.ch.fill) + ", " + lit64(cn.lo) + ", " + lit64(cn.hi) + ", " + lit64(cn.map_def) + ", " +
           lit64(cn.map_a) + ", " + lit64(cn.bk_a) + ", " + lit64(cn.M) + ", " + litu64(cn.hs) + ", " +
           i2s(slot[R.src[0]]) + ", " + i2s(R.src[0]) + ", " + i2s(f) + ", " + i2s(q) + ", " + i2s(R.cap[0]) + ", " +
           i2s(R.ncap[0]) + ", " + i2s(cn.mask) + ", " + i2s(cn.null_mask) + ", " + i2s(cn.map_m) + ", " + i2s(cn.bk_m) +
           ", " + i2s(bk_row) + ", " + i2s(mp < 0 ? 0 : mp) + ", " + i2s(f == F - 1 ? 1 : 0) + ", 0},\n";
    }
    if (L.canon.empty()) s += "  {}\n";
    s += "};\n";
    const int K = std::max(1, L.K);
    s += "__constant__ rapk::JLNgram<" + i2s(K) + "> kJN[" + i2s(std::max<size_t>(1, L.units.size())) + "] = {\n";
    for (int q : L.units) {
      const int f = v.perm[q];
      const RbFeat& R = v.feat[f];
      const SProg& pg = v.sprogs[f];
      std::string sl, cp, nc;
      for (int i = 0; i < K; ++i) {
        sl += (i ? ", " : "") + i2s(slot[R.src[i]]);
        cp += (i ? ", " : "") + i2s(R.cap[i]);
        nc += (i ? ", " : "") + i2s(R.ncap[i]);
      }
      s += "  {" + litu64(pg.ng.hsalt) + ", " + lit64(pg.ng.M) + ", " + i2s(f) + ", " + i2s(q) + ", " + i2s(R.out_cap) +
           ", " + i2s(f == F - 1 ? 1 : 0) + ", {" + sl + "}, {" + cp + "}, {" + nc + "}},\n";
    }
    if (L.units.empty()) s += "  {}\n";
    s += "};\n";
    const int NB = std::max<int>(1, (int)L.bk.size());
    s += "__constant__ long long kJL0[" + i2s(NB) + " * 16] = {";
    for (int b = 0; b < NB; ++b)
      for (int k = 0; k < 16; ++k) {
        long long x = INT64_MAX;
        if (b < (int)L.bk.size()) {
          int m = 0;
          for (int f = 0; f < F; ++f)
            if ((v.sprogs[f].cn.mask & CB_BUCKET) && v.sprogs[f].cn.bk_a == L.bk[b]) m = v.sprogs[f].cn.bk_m;
          if (k < m / 64) x = v.itab[L.bk[b] + 64 * k + 63];
        }
        s += (b || k ? ", " : "") + lit64(x);
      }
    s += "};\n";
    s += "__device__ const int64_t* const kJS[" + i2s(NB) + "] = {";
    for (int b = 0; b < NB; ++b) {
      std::string nm = "nullptr";
      if (b < (int)L.bk.size()) {
        int m = 0;
        for (int f = 0; f < F; ++f)
          if ((v.sprogs[f].cn.mask & CB_BUCKET) && v.sprogs[f].cn.bk_a == L.bk[b]) m = v.sprogs[f].cn.bk_m;
        nm = sample_table(L.bk[b], m);
      }
      s += (b ? ", " : "") + nm;
    }
    s += "};\n";
    return s;
  }
  std::string emit_loop(const LoopPlan& L) {
    const int NU = (int)L.units.size(), NC = (int)L.canon.size(), K = L.K, N = L.N;
    std::string s;
    s += "    bool ovf = false;\n    unsigned late = 0;\n";
    if (NU > 0) {
      const std::string KS = i2s(K), NS = i2s(N);
      s += "    int64_t pf[" + KS + "];\n#pragma unroll\n    for (int i = 0; i < " + KS +
           "; ++i) pf[i] = jl_prefetch(p, s, kJC[i], r, in);\n";
      s += "#pragma unroll 1\n    for (int u = 0; u < " + i2s(NU) + "; ++u) {\n";
      s += "      int64_t pn[" + KS + "];\n#pragma unroll\n      for (int i = 0; i < " + KS + "; ++i) pn[i] = u + 1 < " +
           i2s(NU) + " ? jl_prefetch(p, s, kJC[(u + 1) * " + KS + " + i], r, in) : 0;\n";
      s += "      int64_t mm[" + KS + "];\n      int32_t ml[" + KS + "];\n";
      s += "#pragma unroll\n      for (int i = 0; i < " + KS + "; ++i) {\n        mm[i] = 0;\n"
           "        jl_canon<kSmall>(p, s, kJC[u * " + KS + " + i], kJL0, kJS, r, wi, lane, in, row, B, pf[i], &mm[i], &ml[i], ovf);\n      }\n";
      s += "      if (jl_ngram<" + KS + ", " + NS + ", kSmall>(p, s, kJN[u], mm, ml, r, wi, lane, in, row, B, ovf)) late |= 1u << u;\n";
      s += "#pragma unroll\n      for (int i = 0; i < " + KS + "; ++i) pf[i] = pn[i];\n    }\n";
    }
    if (NC > NU * K) {
      const std::string b0 = i2s(NU * K);
      s += "    int64_t p1 = jl_prefetch(p, s, kJC[" + b0 + "], r, in);\n";
      s += "#pragma unroll 1\n    for (int k = " + b0 + "; k < " + i2s(NC) + "; ++k) {\n";
      s += "      const int64_t pn = k + 1 < " + i2s(NC) + " ? jl_prefetch(p, s, kJC[k + 1], r, in) : 0;\n";
      s += "      int64_t mdum = 0;\n      int32_t ldum = 0;\n";
      s += "      jl_canon<kSmall>(p, s, kJC[k], kJL0, kJS, r, wi, lane, in, row, B, p1, &mdum, &ldum, ovf);\n";
      s += "      p1 = pn;\n    }\n";
    }
    if (NU > 0) {
      s += "#pragma unroll 1\n    for (int u = 0; u < " + i2s(NU) + "; ++u)\n"
           "      if (__any_sync(0xffffffffu, (late >> u) & 1u)) {  // NGram rows off the register path\n"
           "        int32_t L;\n        long long P0;\n"
           "        jl_ngram_lp<" + i2s(K) + ", " + i2s(N) + ", kSmall>(s, kJN[u], r, wi, lane, in, &L, &P0);\n"
           "        if ((late >> u) & 1u) rb_fallback(p, s, x.slot, kJN[u].f, r, row, L, P0);\n      }\n";
    }
    s += "    if (ovf) atomicExch(c.err, 1);  // values_capacity understated (sp_nnz): nothing stored past it\n";
    return s;
  }

  // ---- batched emitter (default when every output qualifies) ----
  // Outputs are emitted in batches of kBatch in processing order, stage by
  // stage across the batch: (1) lengths, positions, length/offset stores and
  // the pre-MapId stages of every output, (2) every MapId's first two probe
  // slots, (3) MapId selects and SigridHash, (4) Bucketize, (5) the value
  // stores, then the batch's NGram outputs.  Each stage's loads are
  // independent across the batch and the stages are branch-free, so one
  // warp's L2 round trips of a batch overlap instead of queueing output by
  // output (measured: the emit phase tracked one warp's serial chain of
  // ~0.6 us per output).  Rows a MapId resolves only past its first two
  // slots, and NGram rows whose sources are not on the register path, are
  // redone by the generic path after the batches (late rows).
  static int batch_k() { return std::max(1, env_int("RAP_JIT_BATCH", 8)); }
  bool batch_ok() const {
    if (env_int("RAP_JIT_BATCH", 8) == 0 || column_mode()) return false;
    int lates = 0;
    for (int q = 0; q < F; ++q) {
      const int f = v.perm[q];
      const RbFeat& R = v.feat[f];
      const SProg& pg = v.sprogs[f];
      if (R.emit == 0) {
        if (!pg.cn.ok || R.kind != 0 || max_len(f) > 1) return false;
      } else if (R.emit == 3) {
        if (!const_cast<Gen*>(this)->ngram_fast_ok(q)) return false;
        ++lates;
      } else {
        return false;
      }
    }
    return lates <= 32;
  }
  // one canonical stage on x, branch-free: a stage that does not apply to a
  // filled null row (null_mask) keeps the row's value by a select
  std::string sel_stage(const Canon& q, int bit, const std::string& x, const std::string& full,
                        const std::string& expr) {
    if (q.null_mask & bit) return "        " + x + " = " + expr + ";\n";
    return "        " + x + " = " + full + " ? (int64_t)(" + expr + ") : " + x + ";\n";
  }
  std::string bucket_expr(const Canon& q, const std::string& x) {
    if (q.bk_m >= 64 && q.bk_m % 64 == 0 && q.bk_a % 2 == 0) {
      const std::string nm = sample_table(q.bk_a, q.bk_m);
      std::string j0 = "(0";
      for (int k = 0; k < q.bk_m / 64; ++k) j0 += " + (" + x + " >= " + lit64(v.itab[q.bk_a + 64 * k + 63]) + ")";
      j0 += ")";
      const BkTab* t = staged_table(q.bk_a);
      const std::string smp = t ? "reinterpret_cast<const int64_t*>(s.tabs + " + i2s(16 + t->off_s) + ")" : nm;
      const std::string brd = (t && t->off_b >= 0) ? "reinterpret_cast<const int64_t*>(s.tabs + " + i2s(16 + t->off_b) + ")"
                                                   : "c.itab + " + lit64(q.bk_a);
      const std::string fn = !t ? "upper_bound_64" : (t->off_b >= 0 ? "upper_bound_64s" : "upper_bound_64h");
      return fn + "(" + brd + ", " + i2s(q.bk_m) + ", " + smp + ", " + j0 + ", " + x + ")";
    }
    if (q.bk_m >= 64) {
      const std::string nm = sample_table(q.bk_a, q.bk_m);
      return "upper_bound_s8(c.itab + " + lit64(q.bk_a) + ", " + i2s(q.bk_m) + ", " + nm + ", " + i2s(q.bk_m / 8) + ", " + x +
             ")";
    }
    return "upper_bound(c.itab + " + lit64(q.bk_a) + ", " + i2s(q.bk_m) + ", " + x + ")";
  }
  // The value chain of a batch's canonical outputs: v<q> from the prefetched
  // first id pf<q> and the staged row X<q>_0 (declared by the caller), fill,
  // Clamp, MapId (two probe slots, warp-uniform continuation), SigridHash,
  // Bucketize; the NGram word m<f> after the memo stage.
  std::string value_code(const std::vector<int>& canon, const std::vector<char>& is_prov) {
    std::string s;
    for (int q : canon) {
      const int f = v.perm[q];
      const SProg& pg = v.sprogs[f];
      const Canon& cn = pg.cn;
      const std::string Q = i2s(q), Fs = i2s(f), X = "X" + Q + "_0";
      const int ma = is_prov[f] ? memo_point(v.feat[f], cn) : -1;
      s += "    v" + Q + " = " + X + ".valid ? pf" + Q + " : " + lit64(pg.ch.fill) + ";\n";
      if (ma == 16) s += "    m" + Fs + " = v" + Q + ";\n";
      if (cn.mask & CB_CLAMP) {
        s += sel_stage(cn, CB_CLAMP, "v" + Q, X + ".valid",
                       "v" + Q + " < " + lit64(cn.lo) + " ? " + lit64(cn.lo) + " : (v" + Q + " > " + lit64(cn.hi) + " ? " +
                           lit64(cn.hi) + " : v" + Q + ")");
        if (ma == CB_CLAMP) s += "    m" + Fs + " = v" + Q + ";\n";
      }
    }
    for (int q : canon) {
      const Canon& cn = v.sprogs[v.perm[q]].cn;
      if (!(cn.mask & CB_MAPID)) continue;
      s += "    const MapProbe2 pk" + i2s(q) + " = map_first_probe2(c.itab, " + lit64(cn.map_a) + ", " + i2s(cn.map_m) +
           ", v" + i2s(q) + ");\n";
    }
    for (int q : canon) {
      const int f = v.perm[q];
      const Canon& cn = v.sprogs[f].cn;
      const std::string Q = i2s(q), Fs = i2s(f), X = "X" + Q + "_0";
      const int ma = is_prov[f] ? memo_point(v.feat[f], cn) : -1;
      if (cn.mask & CB_MAPID) {
        s += "    { bool mi;\n      int64_t mv = map_sel2(pk" + Q + ", v" + Q + ", " + lit64(cn.map_def) + ", &mi);\n";
        const bool all = (cn.null_mask & CB_MAPID) != 0;
        // rows whose key is past the first two slots probe on (warp-uniform test)
        s += "      if (__any_sync(0xffffffffu, mi)) mv = mi ? map_lookup_from2(c.itab, " + lit64(cn.map_a) + ", " +
             i2s(cn.map_m) + ", " + lit64(cn.map_def) + ", v" + Q + ", pk" + Q + ") : mv;\n";
        s += "      v" + Q + " = " + (all ? "mv" : X + ".valid ? mv : v" + Q) + "; }\n";
        if (ma == CB_MAPID) s += "    m" + Fs + " = v" + Q + ";\n";
      }
      if (cn.mask & CB_SIGRID) {
        s += sel_stage(cn, CB_SIGRID, "v" + Q, X + ".valid",
                       "(int64_t)reduce_M(splitmix_H(" + litu64(cn.hs) + " ^ (uint64_t)v" + Q + "), " + lit64(cn.M) + ")");
        if (ma == CB_SIGRID) s += "    m" + Fs + " = v" + Q + ";\n";
      }
    }
    for (int q : canon) {
      const int f = v.perm[q];
      const Canon& cn = v.sprogs[f].cn;
      const std::string Q = i2s(q), Fs = i2s(f), X = "X" + Q + "_0";
      const int ma = is_prov[f] ? memo_point(v.feat[f], cn) : -1;
      if (cn.mask & CB_BUCKET) {
        s += sel_stage(cn, CB_BUCKET, "v" + Q, X + ".valid", bucket_expr(cn, "v" + Q));
        if (ma == CB_BUCKET) s += "    m" + Fs + " = v" + Q + ";\n";
      }
    }
    return s;
  }
  // Batch 0's canonical outputs of the batched emitter (processing indices).
  std::vector<int> pre_canon() const {
    std::vector<int> c;
    for (int q = 0; q < std::min(F, batch_k()); ++q)
      if (v.feat[v.perm[q]].emit == 0) c.push_back(q);
    return c;
  }
  // pre_emit: batch 0's values before the grid wait (one-chunk blocks), so
  // the wait for the other CTAs' totals and the base loads overlap them.
  bool pre_ok() const {
    return env_int("RAP_JIT_PRE", 1) != 0 && batch_ok() && !pairs() && !pre_canon().empty();
  }
  std::vector<char> prov_flags() const {
    std::vector<char> is_prov(F, 0);
    for (int f = 0; f < F; ++f)
      if (v.feat[f].emit == 0 && v.feat[f].memo_slot >= 0) is_prov[f] = 1;
    return is_prov;
  }
  std::string pre_fn() {
    std::string s;
    if (!pre_ok()) {
      s += "  static constexpr bool kPre = false;\n  struct PreState {};\n";
      s += "  template <class P>\n  static __device__ __forceinline__ PreState pre_emit(const P&, const RbSmem&, const RbCtx&, "
           "int64_t, int) { return PreState{}; }\n";
      return s;
    }
    const std::vector<int> canon = pre_canon();
    const std::vector<char> is_prov = prov_flags();
    s += "  static constexpr bool kPre = true;\n  struct PreState {\n";
    for (int q : canon) {
      s += "    int64_t v" + i2s(q) + ";\n";
      if (is_prov[v.perm[q]]) s += "    int64_t m" + i2s(v.perm[q]) + ";\n";
    }
    s += "  };\n";
    s += "  template <class P>\n  static __device__ __forceinline__ PreState pre_emit(const P& p, const RbSmem& s, "
         "const RbCtx& x, int64_t c0, int nr) {\n" + thread_vars() +
         "    const Common& c = p.c;\n    const bool in = r < nr;\n    (void)c0;\n";
    if (tab_total) s += "    mbar_wait(reinterpret_cast<uint64_t*>(s.tabs), 0u);  // staged tables landed\n";
    for (int q : canon) {
      const RbFeat& R = v.feat[v.perm[q]];
      const std::string Q = i2s(q);
      s += "    int64_t pf" + Q + ";\n    { const RbRow Y" + Q + " = " + rbrow() + "(s, " + i2s(slot[R.src[0]]) +
           ", r);\n      const bool ok = in && Y" + Q + ".valid && Y" + Q + ".b > Y" + Q + ".a;\n      pf" + Q +
           " = rap_ldin(ok ? p.val[" + i2s(R.src[0]) + "] + Y" + Q + ".a : c.itab); }\n";
      s += "    const RbRow X" + Q + "_0 = " + rbrow() + "(s, " + i2s(slot[R.src[0]]) + ", r);\n";
      s += "    int64_t v" + Q + ";\n";
      if (is_prov[v.perm[q]]) s += "    int64_t m" + i2s(v.perm[q]) + " = 0;\n";
    }
    s += value_code(canon, is_prov);
    s += "    PreState ps;\n";
    for (int q : canon) {
      s += "    ps.v" + i2s(q) + " = v" + i2s(q) + ";\n";
      if (is_prov[v.perm[q]]) s += "    ps.m" + i2s(v.perm[q]) + " = m" + i2s(v.perm[q]) + ";\n";
    }
    s += "    return ps;\n  }\n";
    return s;
  }
  std::string emit_batched(int qb, int qe) {
    std::string s;
    s += "    unsigned late = 0;\n    (void)late;\n";
    std::vector<char> is_prov(F, 0);
    for (int q = qb; q < qe; ++q) {
      const int f = v.perm[q];
      if (v.feat[f].emit == 0 && v.feat[f].memo_slot >= 0) is_prov[f] = 1;
    }
    for (int f = 0; f < F; ++f)
      if (is_prov[f]) s += "    int64_t m" + i2s(f) + " = 0;\n    int32_t ml" + i2s(f) + " = 0;\n";
    // late slots: every MapId output and every NGram output
    std::vector<int> late_slot(F, -1), late_q;
    for (int q = qb; q < qe; ++q) {
      const int f = v.perm[q];
      const bool lt = v.feat[f].emit == 3;
      if (lt) {
        late_slot[q] = (int)late_q.size();
        late_q.push_back(q);
      }
    }
    auto prefetch = [&](int q) {
      const RbFeat& R = v.feat[v.perm[q]];
      const std::string Y = "Y" + i2s(q);
      return "    int64_t pf" + i2s(q) + ";\n    { const RbRow " + Y + " = " + rbrow() + "(s, " + i2s(slot[R.src[0]]) +
             ", r);\n      const bool ok = in && " + Y + ".valid && " + Y + ".b > " + Y + ".a;\n      pf" + i2s(q) +
             " = rap_ldin(ok ? p.val[" + i2s(R.src[0]) + "] + " + Y + ".a : c.itab); }\n";
    };
    const int K = batch_k();
    std::vector<std::vector<int>> batches;
    for (int q0 = qb; q0 < qe; q0 += K) {
      std::vector<int> b;
      for (int q = q0; q < std::min(qe, q0 + K); ++q) b.push_back(q);
      batches.push_back(b);
    }
    auto pf_batch = [&](const std::vector<int>& b) {
      std::string t;
      for (int q : b)
        if (v.feat[v.perm[q]].emit == 0) t += prefetch(q);
      return t;
    };
    if (!batches.empty()) {
      if (pre_ok() && qb == 0) {  // batch 0's ids only when its values were not carried over
        for (int q : batches[0])
          if (v.feat[v.perm[q]].emit == 0) s += "    int64_t pf" + i2s(q) + " = 0;\n";
        s += "    if (!use_pre) {\n";
        for (int q : batches[0])
          if (v.feat[v.perm[q]].emit == 0) {
            const RbFeat& R = v.feat[v.perm[q]];
            const std::string Q = i2s(q);
            s += "    { const RbRow Y" + Q + " = " + rbrow() + "(s, " + i2s(slot[R.src[0]]) + ", r);\n      const bool ok = in && Y" + Q +
                 ".valid && Y" + Q + ".b > Y" + Q + ".a;\n      pf" + Q + " = rap_ldin(ok ? p.val[" + i2s(R.src[0]) + "] + Y" + Q +
                 ".a : c.itab); }\n";
          }
        s += "    }\n";
      } else {
        s += pf_batch(batches[0]);
      }
    }
    for (size_t bi = 0; bi < batches.size(); ++bi) {
      const std::vector<int>& b = batches[bi];
      if (bi + 1 < batches.size()) s += pf_batch(batches[bi + 1]);  // the next batch's ids in flight
      s += "  {  // batch of outputs";
      for (int q : b) s += " " + i2s(v.perm[q]);
      s += "\n";
      std::vector<int> canon, ngram;
      for (int q : b) (v.feat[v.perm[q]].emit == 0 ? canon : ngram).push_back(q);
      // (1) lengths, positions, length/offset stores
      for (int q : canon) {
        const int f = v.perm[q];
        const std::string Q = i2s(q), Fs = i2s(f);
        s += len_code(q);
        s += "    const long long P" + Q + " = s.wb[" + i2s(q * 8) + " + wi] + rb_ballot_excl(L" + Q + " != 0, lane);\n";
        if (is_prov[f]) s += "    ml" + Fs + " = L" + Q + ";\n";
        s += "    stg_s32_if(in, c.lengths + ((int64_t)" + Fs + " * B + row), L" + Q + ");\n";
        s += "    stg_s64_if(in, c.offsets + ((int64_t)" + Fs + " * B + row), P" + Q + ");\n";
        if (f == F - 1) s += "    stg_s64_if(in && row == B - 1, c.offsets + (int64_t)" + i2s(F) + " * B, P" + Q + " + L" + Q + ");\n";
        s += "    int64_t v" + Q + ";\n";
      }
      // (2)-(4) the values: computed here, or (batch 0 of a one-chunk block)
      // before the grid wait by pre_emit and carried over in registers
      if (bi == 0 && qb == 0 && pre_ok()) {
        s += "    if (use_pre) {\n";
        for (int q : canon) {
          s += "      v" + i2s(q) + " = ps.v" + i2s(q) + ";\n";
          if (is_prov[v.perm[q]]) s += "      m" + i2s(v.perm[q]) + " = ps.m" + i2s(v.perm[q]) + ";\n";
        }
        s += "    } else {\n" + value_code(canon, is_prov) + "    }\n";
      } else {
        s += value_code(canon, is_prov);
      }
      // (5) value stores
      for (int q : canon) {
        const std::string Q = i2s(q);
        s += "    stv_if(L" + Q + " > 0 && P" + Q + " < c.values_cap, c, P" + Q + ", v" + Q + ");\n";
      }
      // the batch's NGram outputs (their providers' memo words are final)
      for (int q : ngram) {
        const int f = v.perm[q];
        const RbFeat& R = v.feat[f];
        const SProg& pg = v.sprogs[f];
        const std::string Q = i2s(q), Fs = i2s(f);
        const int n = R.n, Kk = R.k;
        s += "  {  // output " + Fs + " (NGram)\n" + len_code(q);
        s += "    const long long P" + Q + " = s.wb[" + i2s(q * 8) + " + wi] + " +
             (max_len(f) <= 1 ? "rb_ballot_excl(L" + Q + " != 0, lane)" : "rb_warp_excl<kSmall>(L" + Q + ", lane)") + ";\n";
        s += "    stg_s32_if(in, c.lengths + ((int64_t)" + Fs + " * B + row), L" + Q + ");\n";
        s += "    stg_s64_if(in, c.offsets + ((int64_t)" + Fs + " * B + row), P" + Q + ");\n";
        if (f == F - 1) s += "    stg_s64_if(in && row == B - 1, c.offsets + (int64_t)" + i2s(F) + " * B, P" + Q + " + L" + Q + ");\n";
        std::string cond;
        for (int i = 0; i < Kk; ++i) {
          const int qp = R.prov[i], fp = v.perm[qp];
          const std::string l = "l" + Q + "_" + i2s(i);
          if (i) cond += " && ";
          cond += "(" + l + " <= 1 && (" + l + " == 0 || ml" + i2s(fp) + " >= 1))";
        }
        s += "    {\n      const bool fast = " + cond + ";\n      int32_t cnt = 0;\n";
        for (int j = 0; j < n; ++j) s += "      uint64_t w" + i2s(j) + " = 0;\n";
        for (int i = 0; i < Kk; ++i) {
          const int fp = v.perm[R.prov[i]];
          const std::string pr = "pr" + i2s(i);
          s += "      const bool " + pr + " = l" + Q + "_" + i2s(i) + " != 0;\n";
          for (int j = 0; j + 1 < n; ++j) s += "      w" + i2s(j) + " = " + pr + " ? w" + i2s(j + 1) + " : w" + i2s(j) + ";\n";
          s += "      w" + i2s(n - 1) + " = " + pr + " ? (uint64_t)m" + i2s(fp) + " : w" + i2s(n - 1) + ";\n";
          s += "      cnt += " + pr + ";\n";
          if (i + 1 >= n) {
            s += "      {\n        uint64_t h = " + litu64(pg.ng.hsalt) + ";\n";
            for (int j = 0; j < n; ++j) s += "        h = splitmix_H(h ^ w" + i2s(j) + ");\n";
            s += "        int64_t v = (int64_t)reduce_M(h, " + lit64(pg.ng.M) + ");\n";
            s += stages(pg.cn, pg.cn.mask, "v", "true", -1, "");
            s += "        const long long at = P" + Q + " + (cnt - " + i2s(n) + ");\n";
            s += "        stv_if(fast && " + pr + " && cnt >= " + i2s(n) + " && cnt - " + i2s(n) + " < L" + Q +
                 " && at < c.values_cap, c, at, v);\n      }\n";
          }
        }
        s += "      if (!fast && L" + Q + " > 0) late |= 1u << " + i2s(late_slot[q]) + ";\n    }\n  }\n";
      }
      s += "  }\n";
      // (experiment knob RAP_JIT_BATCHSYNC: the CTA's warps meet after every
      // batch, so they stream the same window of straight-line code)
      if (env_int("RAP_JIT_BATCHSYNC", 0) && bi + 1 < batches.size())
        s += std::string("    ") + (pairs() ? "__syncthreads();" : (gen_dense_ok() ? "rb_sync<true>();" : "rb_sync<false>();")) + "\n";
    }
    // late rows: the generic path (warp-uniform test per output)
    for (int k = 0; k < (int)late_q.size(); ++k) {
      const int q = late_q[k];
      const int f = v.perm[q];
      const std::string Q = i2s(q), Fs = i2s(f);
      s += "  if (__any_sync(0xffffffffu, (late >> " + i2s(k) + ") & 1u)) {\n" + len_code(q);
      s += "    const long long P" + Q + " = s.wb[" + i2s(q * 8) + " + wi] + " +
           (max_len(f) <= 1 ? "rb_ballot_excl(L" + Q + " != 0, lane)" : "rb_warp_excl<kSmall>(L" + Q + ", lane)") + ";\n";
      s += "    if ((late >> " + i2s(k) + ") & 1u) rb_fallback(p, s, x.slot, " + Fs + ", r, row, L" + Q + ", P" + Q + ");\n  }\n";
    }
    // (values_capacity: checked once per output and block by the skeleton)
    return s;
  }

  std::string emit_body(int qb, int qe) {
    std::string s;
    s += "    bool ovf = false;\n"
         "    unsigned late = 0;\n    (void)late;\n";
    std::vector<int> late_q;
    int n_late = 0;
    // memo registers of the providers
    std::vector<char> is_prov(F, 0);
    for (int q = qb; q < qe; ++q) {
      const int f = v.perm[q];
      if (v.feat[f].emit == 0 && v.feat[f].memo_slot >= 0) is_prov[f] = 1;
    }
    for (int f = 0; f < F; ++f)
      if (is_prov[f]) s += "    int64_t m" + i2s(f) + " = 0;\n    int32_t ml" + i2s(f) + " = 0;\n";
    // first ids of the canonical list outputs, loaded kAhead outputs before
    // their use (the load latency hides under the outputs in between)
    const int kAhead = env_int("RAP_JIT_AHEAD", 4);  // (experiment knob)
    const int kSegment = 1 << 30;  // (barriers every few outputs to keep warps together: measured, no gain)
    std::vector<int> canon_q;
    for (int q = qb; q < qe; ++q)
      if (v.feat[v.perm[q]].emit == 0) canon_q.push_back(q);
    auto prefetch = [&](int q) {
      const RbFeat& R = v.feat[v.perm[q]];
      const std::string Y = "Y" + i2s(q);
      const int sl = slot[R.src[0]];
      std::string t = "    int64_t pf" + i2s(q) + ";\n    { const RbRow " + Y + " = " + rbrow() + "(s, " + i2s(sl) +
                      ", r);\n      const bool ok = in && " + Y + ".valid && " + Y + ".b > " + Y + ".a;\n";
      if (sl < v.id_slots) {
        // the chunk's ids were bulk-copied into shared memory (rb_stage_ids):
        // rows inside the staged range read them there, the rest from global
        t += "      const long long j = (long long)" + Y + ".a - s.ide0[" + i2s(sl) + "];\n"
             "      const bool sh = ok && (unsigned long long)j < (unsigned long long)kRbIdCap;\n"
             "      pf" + i2s(q) + " = sh ? s.ids[" + i2s(sl * kRbIdCap) + " + j] : __ldg(ok && !sh ? p.val[" +
             i2s(R.src[0]) + "] + " + Y + ".a : c.itab); }\n";
        return t;
      }
      // unconditional load (no branch): rows without a first id read a word of the plan blob instead
      return t + "      pf" + i2s(q) + " = rap_ldin(ok ? p.val[" + i2s(R.src[0]) + "] + " + Y + ".a : c.itab); }\n";
    };
    // MapId outputs: their first table probe is loaded kProbe outputs ahead,
    // from the prefetched id run through the stages before MapId
    const int kProbe = env_int("RAP_JIT_PROBE", 2);  // (experiment knob)
    auto has_map = [&](int q) { return (v.sprogs[v.perm[q]].cn.mask & CB_MAPID) != 0; };
    auto probe = [&](int q) {
      const int f = v.perm[q];
      const RbFeat& R = v.feat[f];
      const SProg& pg = v.sprogs[f];
      const Canon& cn = pg.cn;
      const std::string Q = i2s(q), Z = "Z" + Q;
      std::string t = std::string(map2() ? "    MapProbe2 pk" : "    longlong2 pk") + Q + ";\n    { const RbRow " + Z + " = " + rbrow() + "(s, " + i2s(slot[R.src[0]]) +
                      ", r);\n      int64_t u = " + Z + ".valid ? pf" + Q + " : " + lit64(pg.ch.fill) + ";\n";
      t += stages(cn, cn.mask & CB_CLAMP, "u", Z + ".valid", -1, "");
      t += "      pk" + Q + " = " + (map2() ? "map_first_probe2" : "map_first_probe") + "(c.itab, " + lit64(cn.map_a) + ", " + i2s(cn.map_m) + ", u); }\n";
      return t;
    };
    if (env_int("RAP_JIT_SKIP", 0) & 16) return s + "  }\n";  // (experiment knob: empty emit phase)
    for (int i = 0; i < (int)canon_q.size() && i < kAhead; ++i) s += prefetch(canon_q[i]);
    for (int i = 0; i < (int)canon_q.size() && i < kProbe; ++i)
      if (has_map(canon_q[i])) s += probe(canon_q[i]);
    int canon_i = 0;
    for (int q = qb; q < qe; ++q) {
      const int f = v.perm[q];
      const RbFeat& R = v.feat[f];
      const SProg& pg = v.sprogs[f];
      const std::string Q = i2s(q), Fs = i2s(f);
      if (R.emit == 0) {
        if (canon_i + kAhead < (int)canon_q.size()) s += prefetch(canon_q[canon_i + kAhead]);
        if (canon_i + kProbe < (int)canon_q.size() && has_map(canon_q[canon_i + kProbe]))
          s += probe(canon_q[canon_i + kProbe]);
        ++canon_i;
      }
      // branch-free block: every value is computed for every lane, the
      // stores are predicated (lanes past the chunk, empty rows), so the
      // scheduler interleaves neighbouring outputs
      const bool le1 = max_len(f) <= 1;  // every row holds at most one id: ballot scan
      // every kSegment outputs the sparse warps meet, so they run through the
      // straight-line code together (the active window stays in the I-cache)
      if (q > 0 && q % kSegment == 0)
        s += std::string("    ") + (gen_dense_ok() ? "rb_sync<true>();" : "rb_sync<false>();") + "\n";
      s += "  {  // output " + Fs + "\n" + len_code(q);
      s += "    const long long P" + Q + " = s.wb[" + i2s(q * 8) + " + wi] + " +
           (le1 ? "rb_ballot_excl(L" + Q + " != 0, lane)" : "rb_warp_excl<kSmall>(L" + Q + ", lane)") + ";\n";
      if (is_prov[f]) s += "    ml" + Fs + " = L" + Q + ";\n";
      s += "    stg_s32_if(in, c.lengths + ((int64_t)" + Fs + " * B + row), L" + Q + ");\n";
      s += "    stg_s64_if(in, c.offsets + ((int64_t)" + Fs + " * B + row), P" + Q + ");\n";
      if (f == F - 1) s += "    stg_s64_if(in && row == B - 1, c.offsets + (int64_t)" + i2s(F) + " * B, P" + Q + " + L" + Q + ");\n";
      s += "    ovf |= P" + Q + " + L" + Q + " > c.values_cap;\n";
      if (R.emit == 0) {
        const Canon& cn = pg.cn;
        const std::string X = "X" + Q + "_0";
        const int col = R.src[0];
        s += "    {\n        int64_t v = " + X + ".valid ? pf" + Q + " : " + lit64(pg.ch.fill) + ";\n";
        s += stages(cn, cn.mask, "v", X + ".valid", is_prov[f] ? memo_point(R, cn) : -1, "m" + Fs,
                    (cn.mask & CB_MAPID) ? "pk" + Q : "");
        s += "        stv_if(L" + Q + " > 0 && P" + Q + " < c.values_cap, c, P" + Q + ", v);\n";
        if (R.cap[0] > 1) {
          s += "        for (int32_t j = 1; j < L" + Q + "; ++j) {\n";
          s += "          int64_t w = __ldg(p.val[" + i2s(col) + "] + " + X + ".a + j);\n";
          s += stages(cn, cn.mask, "w", "true", -1, "");
          s += "          rb_store(c, P" + Q + " + j, w);\n        }\n";
        }
        s += "    }\n";
      } else if (R.emit == 3 && (env_int("RAP_JIT_SKIP", 0) & 8)) {
        // (experiment knob: NGram ids left out)
      } else if (R.emit == 3 && ngram_fast_ok(q)) {
        // every source memoised by an earlier provider: the present elements
        // shift through an n-register window (selects, R7); rows whose sources
        // hold more than one id run the generic path
        const int n = R.n, K = R.k;
        std::string cond;
        for (int i = 0; i < K; ++i) {
          const int fp = v.perm[R.prov[i]];
          const std::string l = "l" + Q + "_" + i2s(i);
          if (i) cond += " && ";
          cond += "(" + l + " <= 1 && (" + l + " == 0 || ml" + i2s(fp) + " >= 1))";
        }
        s += "    {\n      const bool fast = " + cond + ";\n      int32_t cnt = 0;\n";
        for (int j = 0; j < n; ++j) s += "      uint64_t w" + i2s(j) + " = 0;\n";
        for (int i = 0; i < K; ++i) {
          const int fp = v.perm[R.prov[i]];
          const std::string pr = "pr" + i2s(i);
          s += "      const bool " + pr + " = l" + Q + "_" + i2s(i) + " != 0;\n";
          for (int j = 0; j + 1 < n; ++j)
            s += "      w" + i2s(j) + " = " + pr + " ? w" + i2s(j + 1) + " : w" + i2s(j) + ";\n";
          s += "      w" + i2s(n - 1) + " = " + pr + " ? (uint64_t)m" + i2s(fp) + " : w" + i2s(n - 1) + ";\n";
          s += "      cnt += " + pr + ";\n";
          if (i + 1 >= n) {
            s += "      {\n        uint64_t h = " + litu64(pg.ng.hsalt) + ";\n";
            for (int j = 0; j < n; ++j) s += "        h = splitmix_H(h ^ w" + i2s(j) + ");\n";
            s += "        int64_t v = (int64_t)reduce_M(h, " + lit64(pg.ng.M) + ");\n";
            s += stages(pg.cn, pg.cn.mask, "v", "true", -1, "");
            s += "        const long long at = P" + Q + " + (cnt - " + i2s(n) + ");\n";
            s += "        stv_if(fast && " + pr + " && cnt >= " + i2s(n) + " && cnt - " + i2s(n) + " < L" + Q +
                 " && at < c.values_cap, c, at, v);\n      }\n";
          }
        }
        if (n_late < 32) {  // rows the register path cannot take: after the straight-line code
          s += "      if (!fast && L" + Q + " > 0) late |= 1u << " + i2s(n_late) + ";\n    }\n";
          late_q.push_back(q);
          ++n_late;
        } else {
          s += "      if (!fast && L" + Q + " > 0) rb_fallback(p, s, x.slot, " + Fs + ", r, row, L" + Q + ", P" + Q +
               ");\n    }\n";
        }
      } else if (R.emit == 3) {
        s += "    if (L" + Q + " > 0) rb_fallback(p, s, x.slot, " + Fs + ", r, row, L" + Q + ", P" + Q + ");\n";
      } else {
        s += "    if (L" + Q + " > 0) rb_fallback(p, s, x.slot, " + Fs + ", r, row, L" + Q + ", P" + Q + ");\n";
      }
      s += "  }\n";
    }
    for (int k = 0; k < (int)late_q.size(); ++k) {  // NGram rows off the register path (warp-uniform test)
      const int q = late_q[k];
      const std::string Q = i2s(q), Fs = i2s(v.perm[q]);
      s += "  if (__any_sync(0xffffffffu, (late >> " + i2s(k) + ") & 1u)) {\n" + len_code(q);
      s += "    const long long P" + Q + " = s.wb[" + i2s(q * 8) + " + wi] + rb_warp_excl<kSmall>(L" + Q + ", lane);\n";
      s += "    if ((late >> " + i2s(k) + ") & 1u) rb_fallback(p, s, x.slot, " + Fs + ", r, row, L" + Q + ", P" + Q +
           ");\n  }\n";
    }
    s += "    if (ovf) atomicExch(c.err, 1);  // values_capacity understated (sp_nnz): nothing stored past it\n";
    return s;
  }

  // ---- column emitter (RAP_JIT_EMIT=col; measured slower, kept for the record) ----
  // Each sparse warp runs a static, cost-balanced list of outputs; for one
  // output it loops over the chunk's row groups (32 rows each), so a warp
  // re-executes one short output body (its immediates included) instead of
  // streaming every output's code once -- the straight-line row emitter's
  // code (~200 KB for C2) missed the instruction caches (ncu: no_instruction
  // was the top stall of phase 4).  NGram sources memoised by their provider
  // outputs go through shared memory: providers run first, one named barrier,
  // then the NGram outputs.  Ids are loaded two row groups ahead and MapId's
  // first probe one ahead.  Measured on C2 (B200, 65536 rows): phase 4 took
  // 49.7 us against the row emitter's 21.3 us -- the row emitter's cross-output
  // instruction-level parallelism outweighs its instruction-cache misses
  // (a unit's row groups form one dependent chain per warp).
  static bool column_mode() {
    const char* e = getenv("RAP_JIT_EMIT");  // "col": this emitter (experiment knob)
    return e && strcmp(e, "col") == 0;
  }
  int sparse_warps() const { return gen_dense_ok() ? 7 : 8; }
  int memo_off() const { return gen_dense_ok() ? ((tile_offset() + 32 * pitch() * 4 + 15) & ~15) : 0; }
  std::vector<int> col_memo;  // output f -> its memo row in column mode (-1: none)
  int col_memo_slots() {
    col_memo.assign(F, -1);
    int n = 0;
    for (int f = 0; f < F; ++f)
      if (v.feat[f].emit == 0 && v.feat[f].memo_slot >= 0) col_memo[f] = n++;
    return n;
  }
  // shared-memory bytes of region 0 the column emitter needs (0: no memo)
  int dense_need() {
    if (!column_mode()) return 0;
    const int n = col_memo_slots();
    return n ? memo_off() + n * kRbChunk * 8 : 0;
  }
  double out_cost(int q) const {
    const int f = v.perm[q];
    const RbFeat& R = v.feat[f];
    const Canon& cn = v.sprogs[f].cn;
    if (R.emit == 0) {
      double c = 1.0;
      if (cn.mask & CB_MAPID) c += 0.7;
      if (cn.mask & CB_BUCKET) c += 0.5;
      if (R.cap[0] > 1) c += 1.0;
      return c;
    }
    if (R.emit == 3) return 0.6 + 0.5 * R.k + 0.6 * std::max(1, R.k - R.n + 1) * R.n;
    return 4.0;
  }
  // Work units (output q, row groups [g0, g1)) of one phase over nw warps:
  // each output split into k row-group ranges, k the smallest in {1, 2, 3, 4,
  // 7} whose longest-processing-time assignment is within 8% of the mean load
  // (a few NGram outputs over 7 warps need splitting; many outputs do not).
  struct Unit {
    int q, g0, g1;
  };
  std::vector<std::vector<Unit>> assign(const std::vector<int>& qs, int nw) const {
    const int nrg = sparse_warps();
    std::vector<std::vector<Unit>> best;
    double best_ratio = 1e30;
    for (int k : {1, 2, 3, 4, 7}) {
      if (k > nrg) break;
      std::vector<std::pair<double, Unit>> units;
      double total = 0;
      for (int q : qs)
        for (int i = 0; i < k; ++i) {
          const int g0 = nrg * i / k, g1 = nrg * (i + 1) / k;
          const double c = out_cost(q) * (g1 - g0) / nrg + 0.15;  // + the pipeline warm-up of a unit
          units.push_back({c, Unit{q, g0, g1}});
          total += c;
        }
      std::stable_sort(units.begin(), units.end(), [](const auto& a, const auto& b) { return a.first > b.first; });
      std::vector<std::vector<Unit>> w(nw);
      std::vector<double> load(nw, 0.0);
      for (const auto& u : units) {
        const int j = (int)(std::min_element(load.begin(), load.end()) - load.begin());
        w[j].push_back(u.second);
        load[j] += u.first;
      }
      const double ratio = *std::max_element(load.begin(), load.end()) / (total / nw);
      if (ratio < best_ratio) {
        best_ratio = ratio;
        best = w;
      }
      if (ratio <= 1.08) break;
    }
    for (auto& l : best)  // processing order inside a warp
      std::sort(l.begin(), l.end(), [](const Unit& a, const Unit& b) { return a.q != b.q ? a.q < b.q : a.g0 < b.g0; });
    return best;
  }
  // the row-group loop of one output over row groups [g0, g1)
  std::string col_output(int q, int g0, int g1) {
    const int f = v.perm[q];
    const RbFeat& R = v.feat[f];
    const SProg& pg = v.sprogs[f];
    const std::string Q = i2s(q), Fs = i2s(f);
    const int nrg = sparse_warps();
    const bool le1 = max_len(f) <= 1;
    std::string s = "  {  // output " + Fs + ", row groups " + i2s(g0) + ".." + i2s(g1 - 1) + "\n";
    const bool canon = R.emit == 0;
    const bool map = canon && (pg.cn.mask & CB_MAPID);
    if (canon) {
      const std::string sl = i2s(slot[R.src[0]]), col = i2s(R.src[0]);
      s += "    auto ld = [&](int g2) -> int64_t {\n"
           "      const int r2 = min(g2 * 32 + lane, " + i2s(kRbChunk - 1) + ");\n"
           "      const RbRow Y = rb_row(s, " + sl + ", r2);\n"
           "      return __ldg(r2 < nr && Y.valid && Y.b > Y.a ? p.val[" + col + "] + Y.a : c.itab);\n    };\n";
      s += "    int64_t pfA = ld(" + i2s(g0) + "), pfB = ld(" + i2s(g0 + 1) + ");\n";
      if (map) {
        s += "    auto pr = [&](int g2, int64_t id) -> longlong2 {\n"
             "      const int r2 = min(g2 * 32 + lane, " + i2s(kRbChunk - 1) + ");\n"
             "      const RbRow Z = rb_row(s, " + sl + ", r2);\n"
             "      int64_t u = Z.valid ? id : " + lit64(pg.ch.fill) + ";\n";
        s += stages(pg.cn, pg.cn.mask & CB_CLAMP, "u", "Z.valid", -1, "");
        s += "      return map_first_probe(c.itab, " + lit64(pg.cn.map_a) + ", " + i2s(pg.cn.map_m) + ", u);\n    };\n";
        s += "    longlong2 pkA = pr(" + i2s(g0) + ", pfA);\n";
      }
    }
    (void)nrg;
    s += "#pragma unroll 1\n    for (int rg = " + i2s(g0) + "; rg < " + i2s(g1) + " && rg * 32 < nr; ++rg) {\n"
         "    const int r = rg * 32 + lane;\n    const bool in = r < nr;\n    const int64_t row = c0 + r;\n";
    if (canon) {
      s += "    const int64_t pf" + Q + " = pfA;\n    pfA = pfB;\n    pfB = ld(rg + 2);\n";
      if (map) s += "    const longlong2 pk" + Q + " = pkA;\n    pkA = pr(rg + 1, pfA);\n";
    }
    s += len_code(q);
    s += "    const long long P" + Q + " = s.wb[" + i2s(q * 8) + " + rg] + " +
         (le1 ? "rb_ballot_excl(L" + Q + " != 0, lane)" : "rb_warp_excl<kSmall>(L" + Q + ", lane)") + ";\n";
    s += "    stg_s32_if(in, c.lengths + ((int64_t)" + Fs + " * B + row), L" + Q + ");\n";
    s += "    stg_s64_if(in, c.offsets + ((int64_t)" + Fs + " * B + row), P" + Q + ");\n";
    if (f == F - 1) s += "    stg_s64_if(in && row == B - 1, c.offsets + (int64_t)" + i2s(F) + " * B, P" + Q + " + L" + Q + ");\n";
    s += "    ovf |= P" + Q + " + L" + Q + " > c.values_cap;\n";
    if (canon) {
      const Canon& cn = pg.cn;
      const std::string X = "X" + Q + "_0";
      const int col = R.src[0];
      const bool prov = col_memo[f] >= 0;
      s += "    {\n        int64_t v = " + X + ".valid ? pf" + Q + " : " + lit64(pg.ch.fill) + ";\n";
      if (prov) s += "        int64_t mv = 0;\n";
      s += stages(cn, cn.mask, "v", X + ".valid", prov ? memo_point(R, cn) : -1, "mv", map ? "pk" + Q : "");
      if (prov) s += "        memo[" + i2s(col_memo[f] * kRbChunk) + " + r] = mv;\n";
      s += "        stv_if(L" + Q + " > 0 && P" + Q + " < c.values_cap, c, P" + Q + ", v);\n";
      if (R.cap[0] > 1) {
        s += "        for (int32_t j = 1; j < L" + Q + "; ++j) {\n";
        s += "          int64_t w = __ldg(p.val[" + i2s(col) + "] + " + X + ".a + j);\n";
        s += stages(cn, cn.mask, "w", "true", -1, "");
        s += "          rb_store(c, P" + Q + " + j, w);\n        }\n";
      }
      s += "    }\n";
    } else if (R.emit == 3 && col_fast_ok(q)) {
      const int n = R.n, K = R.k;
      // the providers' lengths (whether their memo holds an id) and memo words
      std::vector<int> seen;
      for (int i = 0; i < K; ++i) {
        const int qp = R.prov[i];
        if (std::find(seen.begin(), seen.end(), qp) != seen.end()) continue;
        seen.push_back(qp);
        s += len_code(qp);
        s += "    const int64_t mm" + i2s(qp) + " = memo[" + i2s(col_memo[v.perm[qp]] * kRbChunk) + " + r];\n";
      }
      std::string cond;
      for (int i = 0; i < K; ++i) {
        const std::string l = "l" + Q + "_" + i2s(i);
        if (i) cond += " && ";
        cond += "(" + l + " <= 1 && (" + l + " == 0 || L" + i2s(R.prov[i]) + " >= 1))";
      }
      s += "    {\n      const bool fast = " + cond + ";\n      int32_t cnt = 0;\n";
      for (int j = 0; j < n; ++j) s += "      uint64_t w" + i2s(j) + " = 0;\n";
      for (int i = 0; i < K; ++i) {
        const std::string pr = "pr" + i2s(i);
        s += "      const bool " + pr + " = l" + Q + "_" + i2s(i) + " != 0;\n";
        for (int j = 0; j + 1 < n; ++j)
          s += "      w" + i2s(j) + " = " + pr + " ? w" + i2s(j + 1) + " : w" + i2s(j) + ";\n";
        s += "      w" + i2s(n - 1) + " = " + pr + " ? (uint64_t)mm" + i2s(R.prov[i]) + " : w" + i2s(n - 1) + ";\n";
        s += "      cnt += " + pr + ";\n";
        if (i + 1 >= n) {
          s += "      {\n        uint64_t h = " + litu64(pg.ng.hsalt) + ";\n";
          for (int j = 0; j < n; ++j) s += "        h = splitmix_H(h ^ w" + i2s(j) + ");\n";
          s += "        int64_t v = (int64_t)reduce_M(h, " + lit64(pg.ng.M) + ");\n";
          s += stages(pg.cn, pg.cn.mask, "v", "true", -1, "");
          s += "        const long long at = P" + Q + " + (cnt - " + i2s(n) + ");\n";
          s += "        stv_if(fast && " + pr + " && cnt >= " + i2s(n) + " && cnt - " + i2s(n) + " < L" + Q +
               " && at < c.values_cap, c, at, v);\n      }\n";
        }
      }
      s += "      const bool late = !fast && L" + Q + " > 0;\n"
           "      if (__any_sync(0xffffffffu, late) && late) rb_fallback(p, s, x.slot, " + Fs + ", r, row, L" + Q +
           ", P" + Q + ");\n    }\n";
    } else {
      s += "    if (L" + Q + " > 0) rb_fallback(p, s, x.slot, " + Fs + ", r, row, L" + Q + ", P" + Q + ");\n";
    }
    s += "    }\n  }\n";
    return s;
  }
  // NGram q on the memo path: canonical post stages, every source a raw list
  // whose provider memoises it (column mode: the provider runs in phase A)
  bool col_fast_ok(int q) {
    const int f = v.perm[q];
    const RbFeat& R = v.feat[f];
    const SProg& pg = v.sprogs[f];
    if (!pg.cn.ok || R.n < 1 || R.n > kMaxNgramK) return false;
    for (int i = 0; i < R.k; ++i) {
      if (R.src[i] < 0 || R.prov[i] < 0) return false;
      if (col_memo[v.perm[R.prov[i]]] < 0) return false;
    }
    return true;
  }
  std::string col_emit_fn() {
    col_memo_slots();
    const int nw = sparse_warps();
    std::vector<int> phase_a, phase_b;
    for (int q = 0; q < F; ++q) {
      const int f = v.perm[q];
      (col_memo[f] >= 0 ? phase_a : phase_b).push_back(q);
    }
    bool any_consumer = false;
    for (int q : phase_b) any_consumer |= v.feat[v.perm[q]].emit == 3 && col_fast_ok(q);
    if (!any_consumer) {  // no memo reads: one phase
      phase_a.insert(phase_a.end(), phase_b.begin(), phase_b.end());
      phase_b.clear();
    }
    std::string s;
    s += "  template <bool kSmall, class P>\n"
         "  static __device__ __forceinline__ void emit(const P& p, const RbSmem& s, const RbCtx& x, int64_t c0, "
         "int nr, const PreState&, bool, bool) {\n"
         "    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;\n"
         "    const Common& c = p.c;\n"
         "    const int64_t B = x.B;\n"
         "    long long* memo = reinterpret_cast<long long*>(s.dense + " + i2s(memo_off()) + ");\n"
         "    (void)memo;\n"
         "    bool ovf = false;\n";
    for (int ph = 0; ph < 2; ++ph) {
      const std::vector<int>& qs = ph == 0 ? phase_a : phase_b;
      if (qs.empty()) continue;
      if (ph == 1) s += std::string("    ") + (gen_dense_ok() ? "rb_sync<true>();" : "rb_sync<false>();") +
                        "  // providers' memo words visible\n";
      const auto asg = assign(qs, nw);
      s += "    switch (warp) {\n";
      for (int w = 0; w < nw; ++w) {
        if (asg[w].empty()) continue;
        s += "    case " + i2s(w) + ":\n";
        for (const Unit& u : asg[w]) s += col_output(u.q, u.g0, u.g1);
        s += "    break;\n";
      }
      s += "    default: break;\n    }\n";
    }
    s += "    if (ovf) atomicExch(c.err, 1);  // values_capacity understated (sp_nnz): nothing stored past it\n";
    s += "  }\n";
    return s;
  }

  // NGram q can take the register path: canonical post stages, every source
  // a raw list with a provider processed before it.
  bool ngram_fast_ok(int q) {
    const int f = v.perm[q];
    const RbFeat& R = v.feat[f];
    const SProg& pg = v.sprogs[f];
    if (!pg.cn.ok || R.n < 1 || R.n > kMaxNgramK) return false;
    for (int i = 0; i < R.k; ++i) {
      if (R.src[i] < 0 || R.prov[i] < 0 || R.prov[i] >= q) return false;
      const int fp = v.perm[R.prov[i]];
      if (v.feat[fp].emit != 0 || v.feat[fp].memo_slot < 0) return false;
    }
    return true;
  }

  // variant: bit 0 = 32-bit scans (every offset < 2^31), bit 1 = int32 values (Cast)
  std::string source(int variant) {
    const bool small = (variant & 1) != 0;
    std::string s;
    s += "// generated by rap_jit.cpp for one plan (" + i2s(F) + " sparse outputs)\n";
    s += (variant & 2) ? "#define RAP_VALUES_I32 1\n" : "#define RAP_VALUES_I64 1\n";
    if (env_int("RAP_JIT_STCS", 1)) s += "#define RAP_ST_CS 1\n";  // streaming output stores (rap_rows_skel.cuh)
    if (env_int("RAP_JIT_LDCS", 0)) s += "#define RAP_LD_CS 1\n";  // (experiment knob)
    if (env_int("RAP_JIT_STPLAIN", 0)) s += "#define RAP_ST_PLAIN 1\n";  // (experiment knob)
    s += "#define RAP_BASES_UNROLL " + i2s(env_int("RAP_JIT_BASES_UNROLL", 4)) + "\n";  // (experiment knob)
    if (env_int("RAP_JIT_PREFETCH", 0)) s += "#define RAP_PREFETCH_IDS 1\n";  // (experiment knob)
    s += "#include \"rap_rows_interp.cuh\"\n\nnamespace rapk {\n\n";
    bool records = false;  // does any output fall back to the interpreter's functions?
    for (int f = 0; f < F; ++f) records |= v.feat[f].emit != 0;
    std::string globals;
    const std::string dense = dense_fn(&globals);
    std::string body;
    body += "struct JitPolicy {\n";
    // setup (before phase 1 when tables are staged): the bulk copies of the
    // Bucketize tables, awaited at the start of the emit phase
    body += std::string("  static constexpr bool kSetupEarly = ") + (tab_total ? "true" : "false") + ";\n";
    body += "  static constexpr bool kPairs = " + std::string(pairs() ? "true" : "false") + ";\n";
    body += "  static constexpr int kThreads = " + i2s(threads()) + ";\n";
    body += std::string("  static constexpr bool kPDL = ") + (jit_pdl() ? "true" : "false") + ";\n";
    body += std::string("  static constexpr bool kBasesByDense = ") +
            (dense_mode() == 3 && env_int("RAP_JIT_BASES_DENSE", 0) ? "true" : "false") + ";\n";
    body += std::string("  static constexpr bool kDenseLate = ") +
            (dense_mode() == 3 && env_int("RAP_JIT_DENSE_LATE", 0) ? "true" : "false") + ";\n";
    body += "  template <class P>\n"
            "  static __device__ __forceinline__ void setup(const P& p, const RbSmem& s, const RbCtx& x) {\n";
    (void)records;  // the fallbacks rebuild their record from the plan blob (rb_fallback)
    body += setup_tables();
    body += "  }\n";
    body += pre_fn();
    body += dense;
    body += lengths_fn();
    {
      std::string e = column_mode() ? col_emit_fn() + tail_fn(F) : emit_fn();
      // (experiment knob RAP_JIT_NOSTORE: 1 = no output stores in the emit
      // phase, 2 = values only, 3 = lengths and offsets only; the stored
      // values fold into a sink so the computation stays)
      const int ns = env_int("RAP_JIT_NOSTORE", 0);
      if (ns) {
        auto rep = [&](const std::string& a, const std::string& b) {
          for (size_t i = e.find(a); i != std::string::npos; i = e.find(a, i + b.size())) e.replace(i, a.size(), b);
        };
        const size_t k = e.find("bool ovf = false;");
        if (k != std::string::npos) e.insert(k, "unsigned long long sink = 0;\n    ");
        if (ns == 1 || ns == 3) rep("stv_if(L", "RAP_SINKV(L");
        if (ns == 1 || ns == 2) {
          rep("stg_s32_if(in,", "RAP_SINK(in,");
          rep("stg_s64_if(in,", "RAP_SINK(in,");
        }
        rep("stv_if(fast", "RAP_SINKV(fast");
        if (ns == 2) rep("RAP_SINKV(fast", "stv_if(fast");
        const size_t z = e.rfind("if (ovf) atomicExch");
        e.insert(z, "if (sink == 0x5eed5eedull) c.values[0] = (int64_t)sink;\n    ");
        body += "#define RAP_SINK(q, p, v) (sink ^= (q) ? (unsigned long long)(v) + (unsigned long long)(p) : 0ull)\n";
        body += "#define RAP_SINKV(q, c_, p, v) (sink ^= (q) ? (unsigned long long)(v) + (unsigned long long)(p) : 0ull)\n";
      }
      body += e;
    }
    body += "};\n\n}  // namespace rapk\n\n";
    {
      const LoopPlan lp = loop_plan();
      if (lp.ok) {  // the tables reference the sample tables: generate them first
        const std::string t = loop_tables(lp);
        body = t + body;
      }
    }
    s += globals + sample_globals + "\n" + body;
    // one variant per module: 32-bit scans (every offset < 2^31) or 64-bit
    const char* mb = getenv("RAP_JIT_MINB");  // CTAs per SM the register budget targets (default 2; pairs 4)
    s += "extern \"C\" __global__ void __launch_bounds__(" + i2s(threads()) + ", " + std::string(mb ? mb : "2") +
         ") rap_jit_kernel(const __grid_constant__ "
         "rapk::RbParams<rapk::kRbMaxDense, rapk::kRbMaxCols> p) {\n"
         "  rapk::rows_body<rapk::JitPolicy, rapk::kRbMaxDense, rapk::kRbMaxCols, " +
         std::string(small ? "true" : "false") + ">(p);\n}\n";
    return s;
  }
};

std::mutex g_cache_mu;
std::map<std::string, JitModule*>* g_cache = nullptr;  // per process, never freed (kernels stay loaded)

void put_log(char* log, int cap, const std::string& msg) {
  if (!log || cap <= 0) return;
  snprintf(log, (size_t)cap, "%s", msg.c_str());
}

}  // namespace

namespace {

// NVRTC: the plan source -> sm_100a CUBIN.  false + log on failure.
bool nvrtc_cubin(const std::string& src, std::vector<char>* cubin, std::string* log) {
  nvrtcProgram prog;
  const char* hdrs[] = {kJitHdrInternal, kJitHdrDevice, kJitHdrSkel, kJitHdrInterp};
  const char* names[] = {"rap_internal.h", "rap_device.cuh", "rap_rows_skel.cuh", "rap_rows_interp.cuh"};
  nvrtcResult r = nvrtcCreateProgram(&prog, src.c_str(), "rap_jit_plan.cu", 4, hdrs, names);
  if (r != NVRTC_SUCCESS) {
    *log = std::string("nvrtcCreateProgram: ") + nvrtcGetErrorString(r);
    return false;
  }
  const char* opts[] = {"--gpu-architecture=sm_100a", "-std=c++17", "-lineinfo", "-ftz=false", "-prec-div=true",
                        "-prec-sqrt=true", "-fmad=true", "-default-device"};
  r = nvrtcCompileProgram(prog, (int)(sizeof(opts) / sizeof(opts[0])), opts);
  size_t n = 0;
  nvrtcGetProgramLogSize(prog, &n);
  std::string lg(n, '\0');
  if (n) nvrtcGetProgramLog(prog, &lg[0]);
  if (r != NVRTC_SUCCESS) {
    nvrtcDestroyProgram(&prog);
    *log = "NVRTC compile failed: " + lg.substr(0, 3000);
    return false;
  }
  size_t cn = 0;
  nvrtcGetCUBINSize(prog, &cn);
  cubin->resize(cn);
  nvrtcGetCUBIN(prog, cubin->data());
  nvrtcDestroyProgram(&prog);
  *log = lg;
  return true;
}

}  // namespace

std::string jit_generate(const JitPlanView& v) { return Gen(v).source(1); }

int jit_dense_need(const JitPlanView& v) { return Gen(v).dense_need(); }

int jit_table_bytes(const JitPlanView& v) { return Gen(v).table_bytes(); }

bool jit_compile_only(const std::string& src, std::string* log) {
  std::vector<char> cubin;
  return nvrtc_cubin(src, &cubin, log);
}

JitModule* jit_build(const JitPlanView& v, int variant, char* log, int log_cap) {
  Gen gen(v);
  const std::string src = gen.source(variant);
  {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    if (!g_cache) g_cache = new std::map<std::string, JitModule*>();
    auto it = g_cache->find(src);
    if (it != g_cache->end()) return it->second;
  }
  const auto t0 = std::chrono::steady_clock::now();
  std::vector<char> cubin;
  std::string lg;
  if (!nvrtc_cubin(src, &cubin, &lg)) {
    put_log(log, log_cap, lg);
    return nullptr;
  }
  JitModule* m = new JitModule();
  cudaError_t e = cudaLibraryLoadData(&m->lib, cubin.data(), nullptr, nullptr, 0, nullptr, nullptr, 0);
  if (e == cudaSuccess) e = cudaLibraryGetKernel(&m->k, m->lib, "rap_jit_kernel");
  if (e != cudaSuccess) {
    put_log(log, log_cap, std::string("cudaLibrary: ") + cudaGetErrorString(e));
    delete m;
    return nullptr;
  }
  m->compile_s = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
  std::lock_guard<std::mutex> lk(g_cache_mu);
  auto it = g_cache->find(src);
  if (it != g_cache->end()) return it->second;  // another thread won the race (the loser's module stays loaded)
  (*g_cache)[src] = m;
  return m;
}

double jit_compile_seconds(const JitModule* m) { return m ? m->compile_s : 0.0; }

int jit_occupancy(JitModule* m, int smem_bytes, int threads, int* ctas_per_sm) {
  const void* k = reinterpret_cast<const void*>(m->k);
  const int rc = ensure_dyn_smem(k, smem_bytes);
  if (rc != 0) return rc;
  return (int)cudaOccupancyMaxActiveBlocksPerMultiprocessor(ctas_per_sm, k, threads, smem_bytes);
}

// Same parameter block as rap_rows.cu's kernel (RbParams<kRbMaxDense, kRbMaxCols>).
struct JitParams {
  Common c;
  RbGeom g;
  const float* dense[kRbMaxDense];
  const uint32_t* dvalid[kRbMaxDense];
  const int32_t* off[kRbMaxCols];
  const int64_t* val[kRbMaxCols];
  const uint32_t* svalid[kRbMaxCols];
};

int launch_jit(JitModule* m, const Common& c, const RbGeom& g, const LaunchRaw& raw, int smem_bytes, int threads,
               void* stream) {
  if (raw.n_dense > kRbMaxDense || raw.n_sparse > kRbMaxCols) return (int)cudaErrorInvalidValue;
  const void* k = reinterpret_cast<const void*>(m->k);
  const int rc = ensure_dyn_smem(k, smem_bytes);
  if (rc != 0) return rc;
  JitParams p;
  memset(&p, 0, sizeof(p));
  p.c = c;
  p.g = g;
  for (int i = 0; i < raw.n_dense; ++i) {
    p.dense[i] = raw.dense[i];
    p.dvalid[i] = raw.dvalid ? raw.dvalid[i] : nullptr;
  }
  for (int i = 0; i < raw.n_sparse; ++i) {
    p.off[i] = raw.off[i];
    p.val[i] = raw.val[i];
    p.svalid[i] = raw.svalid ? raw.svalid[i] : nullptr;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(g.n_rb * g.n_fg + g.n_dcta));
  cfg.blockDim = dim3((unsigned)threads);
  cfg.dynamicSmemBytes = smem_bytes;
  cfg.stream = reinterpret_cast<cudaStream_t>(stream);
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  static const int noncoop = env_int("RAP_NONCOOP", 0);  // (experiment knob: launch-cost measurement only)
  static const int pdl = env_int("RAP_JIT_PDL", 0);
  cudaLaunchAttribute attr2[2];
  attr2[0] = attr[0];
  attr2[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr2[1].val.programmaticStreamSerializationAllowed = 1;
  if (pdl && !noncoop) {
    cfg.attrs = attr2;
    cfg.numAttrs = 2;
  } else {
    cfg.numAttrs = noncoop ? 0 : 1;
  }
  void* args[1] = {&p};
  cudaError_t e = cudaLaunchKernelExC(&cfg, k, args);
  if (e != cudaSuccess) return (int)e;
  return (int)cudaGetLastError();
}

}  // namespace rapk
