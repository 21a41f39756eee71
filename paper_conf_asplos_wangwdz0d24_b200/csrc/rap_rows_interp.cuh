// rap_rows_interp.cuh — the built-in policy of the row-block kernel: every
// output of a feature group is interpreted from its shared-memory record
// (rap_rows_skel.cuh), with canonical chains specialised by stage mask.
// Operator semantics: DESIGN.md §3 readings R1-R20 (Table 1).
#pragma once
#include "rap_rows_skel.cuh"

namespace rapk {

// Closed-form output length of local row r (R5 FirstX cap, R7 NGram count,
// R10 filled null = 1 id, R14 null = empty).
__device__ __forceinline__ int32_t rb_len(const RbF& F, const RbSmem& s, int r) {
  const int kind = F.kind;
  if (kind == 0) {
    const RbRow x = rb_row(s, F.slot[0], r);
    return x.valid ? min(max(x.b - x.a, 0), F.cap[0]) : F.ncap[0];
  }
  if (kind == 1) return F.out_cap;
  long long tot = 0;
  const int k = F.k;
  for (int i = 0; i < k; ++i) {
    const int sl = F.slot[i];
    if (sl < 0) {
      tot += F.cap[i];
      continue;
    }
    const RbRow x = rb_row(s, sl, r);
    tot += x.valid ? min(max(x.b - x.a, 0), F.cap[i]) : F.ncap[i];
  }
  return (int32_t)min(max(tot - (long long)F.n + 1, 0ll), (long long)F.out_cap);
}

__device__ __forceinline__ int32_t rb_len_cached(const RbF& F, const RbSmem& s, int fl, int r) {
  const uint32_t c = s.len[fl * kRbChunk + r];
  return c < kLenBig ? (int32_t)c : rb_len(F, s, r);
}

// Lengths of every output of the group for the staged chunk -> s.len, and
// their warp sums -> s.ws (accumulated over chunks when acc).
template <bool kSmall>
__device__ __forceinline__ void rb_lengths(const RbSmem& s, int FL, int nr, bool acc) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const bool in = tid < nr;
  for (int fl = 0; fl < FL; ++fl) {
    const int32_t len = in ? rb_len(s.feat[fl], s, tid) : 0;
    s.len[fl * kRbChunk + tid] = (uint16_t)min((uint32_t)len, kLenBig);
    const long long w = rb_warp_sum<kSmall>(len);
    if (lane == 0) s.ws[fl * 8 + warp] = acc ? s.ws[fl * 8 + warp] + w : w;
  }
}

// Element 0 of a canonical list output's row (valid: the first child id;
// filled null: the fill), loaded one output ahead of its use.
template <class P>
__device__ __forceinline__ int64_t rb_prefetch(const P& p, const RbSmem& s, int fl, int r, bool in) {
  const RbF& F = s.feat[fl];
  if (F.emit != 0) return 0;
  const int sl = F.slot[0];
  const int32_t a = s.off[sl * s.pitch + r];
  const bool valid = (s.bm[sl * 8 + (r >> 5)] >> (r & 31)) & 1u;
  if (in && valid && s.len[fl * kRbChunk + r] != 0) return __ldg(p.val[F.src0] + a);
  return F.fill;
}

// One element of an NGram source chain (k-th source of program pg) for the
// generic path: element j of the row (start >= 0 valid list, -1 filled null,
// -2 dense bucket).
template <class P>
__device__ __noinline__ int64_t rb_src_elem(const P& p, const SProg& pg, int kk, int32_t start, int64_t row,
                                            int32_t j) {
  const Canon& q = pg.src_cn[kk];
  const Chain& ch = pg.src[kk];
  if (q.ok && start >= -1) {
    int64_t v = start >= 0 ? __ldg(p.val[ch.src] + start + j) : ch.fill;
    canon_part(q, 0xff, p.c.itab, v, start >= 0);
    return v;
  }
  return src_value(p, prog_ops(pg, p.c.ops), pg.tab_off, ch, start, row, j);
}

// Generic list (non-canonical chain) or dense Bucketize output.
template <class P>
__device__ __noinline__ void rb_emit_generic(const P& p, const RbSmem s, const RbF& F, int r, int64_t row,
                                             int32_t len, long long pos) {
  const SProg& pg = p.c.sprogs[F.f];
  const DevOp* ops = prog_ops(pg, p.c.ops);
  if (F.emit == 2) {  // dense Bucketize (R4): one id
    if (len > 0) rb_store(p.c, pos, src_value(p, ops, pg.tab_off, pg.ch, -2, row, 0));
    return;
  }
  const RbRow x = rb_row(s, F.slot[0], r);
  const int32_t start = x.valid ? x.a : -1;
  for (int32_t j = 0; j < len; ++j) rb_store(p.c, pos + j, src_value(p, ops, pg.tab_off, pg.ch, start, row, j));
}

// Canonical chain with its stage set MASK fixed at compile time: Clamp (R6)
// -> MapId (R8) -> SigridHash (R1-R3) -> Bucketize (R4), parameters read
// from the shared-memory record.  A stage runs on a filled null row (full =
// false) only if it follows the FillNull (null_mask, R10).  Element 0 is
// memoised after stage bit memo_after (16: before the first stage).
template <int MASK>
__device__ __forceinline__ int64_t canon_run(const Canon& q, const int64_t* itab, int64_t v, bool full,
                                             int memo_after, long long* memo) {
  const int nmask = q.null_mask;
  if (memo_after == 16) *memo = v;
  if (MASK & CB_CLAMP) {
    if (full || (nmask & CB_CLAMP)) {
      const int64_t lo = q.lo, hi = q.hi;
      v = v < lo ? lo : v;
      v = v > hi ? hi : v;
    }
    if (memo_after == CB_CLAMP) *memo = v;
  }
  if (MASK & CB_MAPID) {
    if (full || (nmask & CB_MAPID)) v = map_lookup(itab, q.map_a, q.map_m, q.map_def, 0, 0, v);
    if (memo_after == CB_MAPID) *memo = v;
  }
  if (MASK & CB_SIGRID) {
    if (full || (nmask & CB_SIGRID)) v = (int64_t)reduce_M(splitmix_H(q.hs ^ (uint64_t)v), q.M);
    if (memo_after == CB_SIGRID) *memo = v;
  }
  if (MASK & CB_BUCKET) {
    if (full || (nmask & CB_BUCKET)) v = upper_bound(itab + q.bk_a, q.bk_m, v);
    if (memo_after == CB_BUCKET) *memo = v;
  }
  return v;
}

// Ids of a canonical list output for this thread's row: element 0 (x0) was
// loaded one output ahead; further elements (multi-id rows) load here.
template <int MASK, class P>
__device__ __forceinline__ void emit_canon(const P& p, const RbSmem& s, const RbF& F, int r, int32_t len,
                                           long long pos, int64_t x0) {
  if (len == 0) return;
  const int sl = F.slot[0];
  const bool valid = (s.bm[sl * 8 + (r >> 5)] >> (r & 31)) & 1u;
  const int ms = F.memo_slot;
  long long* memo = s.memo + max(ms, 0) * kRbChunk + r;  // written only when ms >= 0
  const int ma = ms >= 0 ? F.memo_after : -1;
  rb_store(p.c, pos, canon_run<MASK>(F.cn, p.c.itab, x0, valid, ma, memo));
  if (len > 1) {  // only a valid row holds more than one id
    const int32_t a = s.off[sl * s.pitch + r];
    const int64_t* vals = p.val[F.src0] + a;
    for (int32_t j = 1; j < len; ++j)
      rb_store(p.c, pos + j, canon_run<MASK>(F.cn, p.c.itab, __ldg(vals + j), true, -1, memo));
  }
}

template <class P>
__device__ __forceinline__ void emit_canon_any(const P& p, const RbSmem& s, const RbF& F, int r, int32_t len,
                                               long long pos, int64_t x0) {
  switch (F.cn.mask & 15) {
    case 0: emit_canon<0>(p, s, F, r, len, pos, x0); break;
    case 1: emit_canon<1>(p, s, F, r, len, pos, x0); break;
    case 2: emit_canon<2>(p, s, F, r, len, pos, x0); break;
    case 3: emit_canon<3>(p, s, F, r, len, pos, x0); break;
    case 4: emit_canon<4>(p, s, F, r, len, pos, x0); break;
    case 5: emit_canon<5>(p, s, F, r, len, pos, x0); break;
    case 6: emit_canon<6>(p, s, F, r, len, pos, x0); break;
    case 7: emit_canon<7>(p, s, F, r, len, pos, x0); break;
    case 8: emit_canon<8>(p, s, F, r, len, pos, x0); break;
    case 9: emit_canon<9>(p, s, F, r, len, pos, x0); break;
    case 10: emit_canon<10>(p, s, F, r, len, pos, x0); break;
    case 11: emit_canon<11>(p, s, F, r, len, pos, x0); break;
    case 12: emit_canon<12>(p, s, F, r, len, pos, x0); break;
    case 13: emit_canon<13>(p, s, F, r, len, pos, x0); break;
    case 14: emit_canon<14>(p, s, F, r, len, pos, x0); break;
    default: emit_canon<15>(p, s, F, r, len, pos, x0); break;
  }
}

// NGram fast path (R7) for a row whose sources each hold at most one id and
// whose providers memoised it earlier in this CTA: the present elements are
// pushed through a WN-register window, a window of n hashes is emitted per
// element from the n-th on.  Returns false (nothing stored) otherwise.
template <int WN, class P>
__device__ __forceinline__ bool ngram_fast(const P& p, const RbSmem& s, const RbF& F, int fl, int pb, int r,
                                           int32_t len, long long pos, uint64_t hs0, int64_t M) {
  const int n = F.n, K = F.k;
  bool ok = true;
  for (int kk = 0; kk < K; ++kk) {
    const int pv = F.prov[kk];
    const int sl = F.slot[kk];
    if (pv < pb || pv >= pb + fl || sl < 0) return false;
    const RbRow x = rb_row(s, sl, r);
    const int32_t lk = x.valid ? min(max(x.b - x.a, 0), F.cap[kk]) : F.ncap[kk];
    ok &= lk <= 1 && (lk == 0 || s.len[(pv - pb) * kRbChunk + r] >= 1);
  }
  if (!ok) return false;
  uint64_t w[WN];
#pragma unroll
  for (int i = 0; i < WN; ++i) w[i] = 0;
  int32_t cnt = 0;
  for (int kk = 0; kk < K; ++kk) {
    const int sl = F.slot[kk];
    const RbRow x = rb_row(s, sl, r);
    const int32_t lk = x.valid ? min(max(x.b - x.a, 0), F.cap[kk]) : F.ncap[kk];
    if (lk == 0) continue;
    const uint64_t e = (uint64_t)s.memo[F.pslot[kk] * kRbChunk + r];
#pragma unroll
    for (int i = 0; i < WN - 1; ++i) w[i] = w[i + 1];
    w[WN - 1] = e;
    ++cnt;
    if (cnt >= n && cnt - n < len) {
      uint64_t h = hs0;
#pragma unroll
      for (int i = 0; i < WN; ++i)
        if (i >= WN - n) h = splitmix_H(h ^ w[i]);
      int64_t v = (int64_t)reduce_M(h, M);
      if (F.cn.mask) canon_part(F.cn, 0xff, p.c.itab, v, true);
      rb_store(p.c, pos + (cnt - n), v);
    }
  }
  return true;
}

// NGram (R7): c = concatenation of the k source lists; window j hashes
// c[j .. j+n) into H(salt) in order; the post ops run on reduce(h, M).
// A source whose provider ran earlier in this CTA reads its memoised
// element 0 (rows with at most one id); anything else is recomputed.
template <class P>
__device__ __noinline__ void rb_emit_ngram(const P& p, const RbSmem s, const RbF& F, int fl, int r, int64_t row,
                                           int32_t len, long long pos, int pb) {
  const SProg& pg = p.c.sprogs[F.f];
  const int n = F.n, K = F.k;
  const uint64_t hs0 = pg.ng.hsalt;
  const int64_t M = pg.ng.M;
  uint64_t w[kMaxNgramK];  // the last n elements, w[kMaxNgramK - 1] newest
#pragma unroll
  for (int i = 0; i < kMaxNgramK; ++i) w[i] = 0;
  int32_t cnt = 0;
  for (int kk = 0; kk < K && cnt - n + 1 < len; ++kk) {
    const int sl = F.slot[kk];
    int32_t lk, start;
    if (sl < 0) {
      lk = F.cap[kk];
      start = -2;
    } else {
      const RbRow x = rb_row(s, sl, r);
      lk = x.valid ? min(max(x.b - x.a, 0), F.cap[kk]) : F.ncap[kk];
      start = x.valid ? x.a : -1;
    }
    const int pv = F.prov[kk];
    const bool memo = pv >= pb && pv < pb + fl && lk <= 1 && (lk == 0 || s.len[(pv - pb) * kRbChunk + r] >= 1);
    const int ps = memo ? F.pslot[kk] : 0;
    for (int32_t j = 0; j < lk && cnt - n + 1 < len; ++j) {
      const int64_t e = memo ? s.memo[ps * kRbChunk + r] : rb_src_elem(p, pg, kk, start, row, j);
#pragma unroll
      for (int i = 0; i < kMaxNgramK - 1; ++i) w[i] = w[i + 1];
      w[kMaxNgramK - 1] = (uint64_t)e;
      ++cnt;
      if (cnt >= n) {
        uint64_t h = hs0;
#pragma unroll
        for (int i = 0; i < kMaxNgramK; ++i)
          if (i >= kMaxNgramK - n) h = splitmix_H(h ^ w[i]);
        int64_t v = (int64_t)reduce_M(h, M);
        if (F.cn.ok)
          canon_part(F.cn, 0xff, p.c.itab, v, true);
        else
          v = apply_id_ops(prog_ops(pg, p.c.ops), p.c.itab, pg.tab_off, v, pg.ch.op_begin, pg.ch.op_end);
        rb_store(p.c, pos + (cnt - n), v);
      }
    }
  }
}


// Rare rows of the generated kernel (an NGram row whose sources hold more
// than one id, a non-canonical chain): the output's record is rebuilt from the
// plan blob (RbFeat, SProg) and the interpreter's functions run (no memo).
template <class P>
__device__ __noinline__ void rb_fallback(const P& p, const RbSmem s, const int16_t* slot_map, int f, int r,
                                         int64_t row, int32_t len, long long pos) {
  const RbFeat& G = p.g.feat[f];
  const SProg& pg = p.c.sprogs[f];
  RbF F;
  F.kind = G.kind;
  F.emit = G.emit;
  F.n = G.n;
  F.k = G.k;
  F.out_cap = G.out_cap;
  F.memo_slot = -1;
  F.memo_mask = 0;
  F.f = f;
  const int kk = F.kind == 1 ? 0 : F.k;
  for (int i = 0; i < kMaxNgramK; ++i) {
    F.cap[i] = G.cap[i];
    F.ncap[i] = G.ncap[i];
    F.slot[i] = (i < kk && G.src[i] >= 0) ? slot_map[G.src[i]] : (int16_t)-1;
    F.prov[i] = F.pslot[i] = -1;
  }
  F.fill = pg.ch.fill;
  F.src0 = G.src[0];
  F.memo_after = -1;
  F.cn = pg.cn;
  if (F.emit == 3)
    rb_emit_ngram(p, s, F, -1, r, row, len, pos, 0);
  else
    rb_emit_generic(p, s, F, r, row, len, pos);
}

// The built-in policy: each output's record (RbF) in shared memory, read per
// warp and output.
struct InterpPolicy {
  static constexpr bool kSetupEarly = true;  // the records drive (1) as well
  static constexpr bool kPairs = false;
  static constexpr bool kPre = false;  // (the generated policy's pre_emit: rap_jit.cpp)
  static constexpr bool kDenseLate = false;
  static constexpr bool kBasesByDense = false;
  static constexpr bool kPDL = false;
  static constexpr bool kTail = false;  // (the generated policy's dense-warp tail)
  template <bool kSmall, class P>
  static __device__ __forceinline__ void emit_tail(const P&, const RbSmem&, const RbCtx&, int64_t, int, int) {}
  struct PreState {};
  template <class P>
  static __device__ __forceinline__ PreState pre_emit(const P&, const RbSmem&, const RbCtx&, int64_t, int) {
    return PreState{};
  }
  static constexpr int kThreads = kRbChunk;
  static constexpr bool kGenDense = false;
  static constexpr bool kDenseWarp = false;
  template <class P>
  static __device__ __forceinline__ void dense(const P&, const RbSmem&, const RbCtx&) {}
  template <class P>
  static __device__ __forceinline__ void dense_warp(const P&, const RbSmem&, const RbCtx&) {}

  template <class P>
  static __device__ __forceinline__ void setup(const P& p, const RbSmem& s, const RbCtx& x) {
    const int tid = threadIdx.x;
    if (tid >= x.FL) return;
    const RbGeom& g = p.g;
    const int f = x.fidx[tid];
    const RbFeat& G = g.feat[f];
    RbF& R = s.feat[tid];
    R.kind = __ldg(&G.kind);
    R.emit = __ldg(&G.emit);
    R.n = __ldg(&G.n);
    R.k = __ldg(&G.k);
    R.out_cap = __ldg(&G.out_cap);
    R.memo_slot = __ldg(&G.memo_slot);
    R.memo_mask = __ldg(&G.memo_mask);
    R.f = f;
    const int kk = R.kind == 1 ? 0 : R.k;
    for (int i = 0; i < kMaxNgramK; ++i) {
      R.cap[i] = __ldg(&G.cap[i]);
      R.ncap[i] = __ldg(&G.ncap[i]);
      const int src = __ldg(&G.src[i]);
      R.slot[i] = (i < kk && src >= 0) ? x.slot[src] : (int16_t)-1;
      R.prov[i] = (int16_t)__ldg(&G.prov[i]);
      R.pslot[i] = (int16_t)__ldg(&G.pslot[i]);
    }
    const SProg& pg = p.c.sprogs[f];
    R.src0 = __ldg(&G.src[0]);
    R.fill = pg.ch.fill;
    R.cn = pg.cn;
    // memo point: after the last stage of the provider prefix present in the chain
    const int pm = R.memo_mask & R.cn.mask;
    int ma = pm ? 1 : 16;
    while (pm >> 1 >= ma) ma <<= 1;
    R.memo_after = R.memo_slot >= 0 ? ma : -1;
  }

  template <bool kSmall, class P>
  static __device__ __forceinline__ void lengths(const P& p, const RbSmem& s, const RbCtx& x, int nr, bool acc) {
    rb_lengths<kSmall>(s, x.FL, nr, acc);
  }

  template <bool kSmall, class P>
  static __device__ __forceinline__ void emit(const P& p, const RbSmem& s, const RbCtx& x, int64_t c0, int nr,
                                              const PreState&, bool, bool) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const Common& c = p.c;
    const int FL = x.FL, pb = x.pb, F = x.F;
    const int64_t B = x.B;
    const bool in = tid < nr;
    const int64_t row = c0 + tid;
    int64_t nx = rb_prefetch(p, s, 0, tid, in);
    for (int fl = 0; fl < FL; ++fl) {
      const int64_t x0 = nx;
      if (fl + 1 < FL) nx = rb_prefetch(p, s, fl + 1, tid, in);
      const RbF& Fd = s.feat[fl];
      const int32_t len = in ? rb_len_cached(Fd, s, fl, tid) : 0;
      const long long pos = s.wb[fl * 8 + warp] + rb_warp_excl<kSmall>(len, lane);
      if (!in) continue;
      const int f = Fd.f;
      const int64_t oi = (int64_t)f * B + row;
      rb_store_lo(c, oi, len, pos);
      if (f == F - 1 && row == B - 1) stg_s64(c.offsets + (int64_t)F * B, pos + len);
      const int emit = Fd.emit;
      if (emit == 0) {  // canonical list: Clamp -> MapId -> SigridHash -> Bucketize subset
        emit_canon_any(p, s, Fd, tid, len, pos, x0);
      } else if (emit == 3) {
        if (len > 0) {
          const SProg& pg = c.sprogs[f];
          const uint64_t hs0 = pg.ng.hsalt;
          const int64_t M = pg.ng.M;
          const bool done = Fd.n <= 4 ? ngram_fast<4>(p, s, Fd, fl, pb, tid, len, pos, hs0, M)
                                      : ngram_fast<8>(p, s, Fd, fl, pb, tid, len, pos, hs0, M);
          if (!done) rb_emit_ngram(p, s, Fd, fl, tid, row, len, pos, pb);
        }
      } else {
        rb_emit_generic(p, s, Fd, tid, row, len, pos);
      }
    }
  }
};

}  // namespace rapk
