// dgr_kernels.cu — sm_100a kernels of the DGR solver iteration (§4.3-4.5).
//
// One iteration k is two kernels (plus the NCCL allreduce of the demand when world > 1):
//
//   KG   per G-cell line (CTA / line): scan of the difference arrays -> demand d (Eq. (10),
//        P:556-564), overflow cost f(d - cap) (Eq. (9), reading Q2), gradient map G = a3 f'(d - cap), and
//        the exclusive prefix S of G along the line; clears the difference arrays.
//   KBF  per tile (CTA / tile of whole nets, see dgr_internal.h):
//          reverse of iteration k:  p(k) recomputed (same Gumbel noise), c_i = dcost/dpi_i from
//            O(1) S differences per segment / turning point gathered from the tile's S window in
//            shared memory, segmented softmax backward, Adam on the path logits;
//          tree level: du_j = (q_j/t)(dq_j - mean_q dq), Adam on the tree logits, q(k+1);
//          forward of iteration k+1: p(k+1) from the new logits, pi = q p, the expected-demand
//            events accumulated in the tile's shared-memory window, flushed once to HBM.
//        The first forward of a dgr_step call and the last reverse run the same kernel with one
//        half switched off (KF / KB).
//
// Nothing here is a dense contraction; the path is bound by memory / L2 traffic, so there are
// no tensor-core instructions by design.
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>

#include "dgr_internal.h"

namespace dgr {

constexpr unsigned kFull = 0xffffffffu;

// Timing knock-outs and per-tile phase clocks (DGR_DEBUG_SKIP bits; results invalid) exist only in
// diagnostic builds (DGR_NVCC_EXTRA=-DDGR_DIAG=1): production code carries no checks for them.
#ifndef DGR_DIAG
#define DGR_DIAG 0
#endif
#define KO(bit) (DGR_DIAG && (P.skip & (bit)))

// DGR_ACCURATE=1: correctly rounded-ish fp32 library functions (expf, logf, sqrtf, IEEE division)
// on the per-candidate path instead of the MUFU approximations (experiment: parity vs speed)
#ifndef DGR_NL_EARLY
#define DGR_NL_EARLY 1   // net level: tree moments loaded before its barrier, tree noise before the Adam chain
#endif
#ifndef DGR_HEAD_SOFTMAX
#define DGR_HEAD_SOFTMAX 1   // softmax shifted by the group head's z (exact maximum only when needed)
#endif
#ifndef DGR_ACCURATE
#define DGR_ACCURATE 0
#endif
#if DGR_ACCURATE
#define FEXP(x) expf(x)
#define FLOG(x) logf(x)
#define FDIV(a, b) ((a) / (b))
#else
#define FEXP(x) __expf(x)
#define FLOG(x) __logf(x)
#define FDIV(a, b) __fdividef(a, b)
#endif

// ------------------------------------------------------------------------------------------
// Counter-based noise: Philox4x32-10 keyed on (seed; idx>>2, k, stream), word idx & 3.
// u = ((r >> 9) + 1/2) 2^-23 is exact in fp32; g = -ln(-ln u) (reading Q7).
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint2 key) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    const uint32_t hi0 = __umulhi(0xD2511F53u, c.x), lo0 = 0xD2511F53u * c.x;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c.z), lo1 = 0xCD9E8D57u * c.z;
    c = make_uint4(hi1 ^ c.y ^ key.x, lo1, hi0 ^ c.w ^ key.y, lo0);
    key.x += 0x9E3779B9u;
    key.y += 0xBB67AE85u;
  }
  return c;
}

// the same generator with the round keys precomputed on the host (KParams::rk, constant bank)
__device__ __forceinline__ uint4 philox_rk(uint4 c, const uint32_t* rk) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    const uint32_t hi0 = __umulhi(0xD2511F53u, c.x), lo0 = 0xD2511F53u * c.x;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c.z), lo1 = 0xCD9E8D57u * c.z;
    c = make_uint4(hi1 ^ c.y ^ rk[2 * r], lo1, hi0 ^ c.w ^ rk[2 * r + 1], lo0);
  }
  return c;
}

// g = -ln(-ln u) from one Philox word (the outer log by MUFU: |error| < 1e-6 on g)
__device__ __forceinline__ float gumbel_word(uint32_t w) {
  const float u = ((float)(w >> 9) + 0.5f) * (1.0f / 8388608.0f);
  return -FLOG(-logf(u));
}

__device__ __forceinline__ float gumbel(uint64_t seed, uint64_t idx, uint32_t k, uint32_t stream) {
  const uint4 r = philox4x32_10(make_uint4((uint32_t)(idx >> 2), (uint32_t)(idx >> 34), k, stream),
                                make_uint2((uint32_t)seed, (uint32_t)(seed >> 32)));
  const uint32_t s = (uint32_t)idx & 3u;
  return gumbel_word(s == 0 ? r.x : (s == 1 ? r.y : (s == 2 ? r.z : r.w)));
}

// Gumbel noise (stream 0) of a tile's noisy candidates: the raw Philox word of each into gp[tile noise
// offset] (each lane turns its own word into g = -ln(-ln u) where it uses it: no conversion is spent
// on the words of a quad that no candidate draws); the tile's runs of
// consecutive global noise indices (NoiseRun), one Philox call per aligned quad of indices (one run:
// the quads spread over the CTA's threads; several: a thread per run piece of at most 4 quads).
// VEC (pipelined tiles, one run): quad q goes whole to gp[4q .. 4q + 3] (one 16-byte store per thread,
// no bank conflicts), so the word of tile noise offset o sits at gp[o + noise_shift(P, T)].
__device__ __forceinline__ int noise_shift(const KParams& P, const TileDesc& T) {
  return T.nrun == 1 ? (int)((P.nid_base + T.nid0) & 3) : 0;
}
template <int NT, bool VEC = false>
__device__ __forceinline__ void tile_noise(const KParams& P, const TileDesc& T, uint32_t k, float* gp) {
  if (T.nrun == 1) {   // one run (nets in the caller's order): its quads spread over the threads
    const int64_t g0 = P.nid_base + T.nid0;
    if (VEC) {
      for (int q = threadIdx.x; q < T.nquad; q += NT) {
        const int64_t c = (g0 >> 2) + q;
        reinterpret_cast<uint4*>(gp)[q] = philox_rk(make_uint4((uint32_t)c, (uint32_t)(c >> 32), k, 0u), P.rk);
      }
    } else {
      for (int q = threadIdx.x; q < T.nquad; q += NT) {
        const int64_t c = (g0 >> 2) + q;
        const uint4 w = philox_rk(make_uint4((uint32_t)c, (uint32_t)(c >> 32), k, 0u), P.rk);
        const uint32_t wd[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int64_t o = c * 4 + i - g0;
          if (o >= 0 && o < T.nnoisy) gp[o] = __uint_as_float(wd[i]);
        }
      }
    }
    return;
  }
  // several runs (nets re-ordered by the plan), cut into pieces within one aligned block of 16 noise
  // indices (at most 4 Philox quads each): a thread per piece
  const int4* R = reinterpret_cast<const int4*>(P.runs) + T.run0;   // {off, len, nid, -}
  for (int ri = threadIdx.x; ri < T.nrun; ri += NT) {
    const int4 r = __ldg(&R[ri]);
    const int64_t g0 = P.nid_base + r.z;
    for (int64_t c = g0 >> 2; c <= (g0 + r.y - 1) >> 2; ++c) {
      const uint4 w = philox_rk(make_uint4((uint32_t)c, (uint32_t)(c >> 32), k, 0u), P.rk);
      const uint32_t wd[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int64_t o = c * 4 + i - g0;
        if (o >= 0 && o < r.y) gp[r.x + o] = __uint_as_float(wd[i]);
      }
    }
  }
}

// ------------------------------------------------------------------------------------------
// Per-lane view of a bundle: which sub-net group / tree / global candidate this lane is.
// ------------------------------------------------------------------------------------------
struct Lane {
  int lane, head, end;
  uint32_t pw, shape, le, gmask, hm, tm;
  bool valid;
  int sub, tree;
  bool single;     // lane of a singleton bundle (lone straight sub-nets: p = 1, no noise)
};

__device__ __forceinline__ void lane_setup(const KParams& P, int b, Lane& L) {
  L.lane = threadIdx.x & 31;
  const int4 bi = __ldg(&P.binfo[b]);
  L.pw = __ldg(&P.pword[(size_t)b * 32 + L.lane]);
  L.shape = L.pw & 7u;
  L.valid = L.shape != kPad;
  L.hm = __ballot_sync(kFull, L.pw & kSubHead);    // pad lanes carry kSubHead: own group each
  L.tm = __ballot_sync(kFull, L.pw & kTreeHead);
  L.le = kFull >> (31 - L.lane);
  L.head = 31 - __clz(L.hm & L.le);
  const uint32_t rest = L.hm & ~L.le;
  L.end = rest ? (__ffs(rest) - 2) : 31;
  L.gmask = (kFull >> (31 - L.end)) & ~((1u << L.head) - 1u);
  L.sub = bi.y + __popc(L.hm & L.le) - 1;
  L.tree = bi.z + (int)((L.pw >> kTreeShift) & kTreeMask);
  L.single = (bi.w & kSingleBundle) != 0;
}

// reduction over the lane's group [head, end]; the result is valid at the head lane
template <typename T, typename Op>
__device__ __forceinline__ T seg_reduce(T v, int lane, int end, Op op) {
#pragma unroll
  for (int off = 1; off < 32; off <<= 1) {
    const T o = __shfl_down_sync(kFull, v, off);
    if (lane + off <= end) v = op(v, o);
  }
  return v;
}

struct Sum {
  template <typename T> __device__ __forceinline__ T operator()(T a, T b) const { return a + b; }
};
struct Max {
  __device__ __forceinline__ float operator()(float a, float b) const { return fmaxf(a, b); }
};

// dq_j in 2^-32 fixed point, accumulated in shared memory as three 32-bit limbs (a 64-bit shared
// atomic is a CAS loop on sm_100): v = hi 2^42 + mid 2^21 + lo with lo, mid in [0, 2^21) (up to 1024
// contributions per tree cannot overflow a limb) and hi = v >> 42 signed; exact for any int64 v.
__device__ __forceinline__ void dq_add(int* dq3, int tree, long long v) {
  int* d = dq3 + 3 * tree;
  atomicAdd(d, (int)(v & 0x1FFFFF));
  atomicAdd(d + 1, (int)((v >> 21) & 0x1FFFFF));
  atomicAdd(d + 2, (int)(v >> 42));
}
__device__ __forceinline__ double dq_get(const int* dq3, int tree) {
  const int* d = dq3 + 3 * tree;
  const long long v = ((long long)d[2] << 42) + ((long long)(unsigned)d[1] << 21) + (long long)(unsigned)d[0];
  return (double)v * kDqInv;
}

__device__ __forceinline__ void red64(long long* p, long long v) {
  if (v != 0) atomicAdd(reinterpret_cast<unsigned long long*>(p), static_cast<unsigned long long>(v));
}

// beta v (v in 2^-24) in the 2^-40 fixed point of the difference arrays: an exact integer product
// when beta is a multiple of 2^-16 (beta_exact; the default 0.25 is), else rounded per event
template <bool EXACT = false>
__device__ __forceinline__ long long beta_fold(const StepArgs& A, long long v) {
  if (EXACT) return v * A.beta_qi;
  return A.beta_exact ? v * A.beta_qi : __double2ll_rn(A.beta_q * (double)v);
}

// red.global.add.u64 unless v == 0, predicated instead of branched (no memory clobber: nothing in
// the kernel reads the global difference arrays back)
__device__ __forceinline__ void red64p(long long* p, long long v) {
  asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.s64 q, %1, 0;\n\t@q red.global.add.u64 [%0], %1;\n\t}" ::"l"(p), "l"(v));
}

// Missing incident edges of G-cell (x, y) at the grid border: 4 - deg(x, y)
__device__ __forceinline__ int border_deficit(int x, int y, int X, int Y) {
  return (x == 0) + (x == X - 1) + (y == 0) + (y == Y - 1);
}

// A turning point at (x, y) with probability weight v (2^-24) adds beta v to each incident edge
// (Eq. (10), reading Q3): edges x-1 and x of row y, y-1 and y of column x (clipped at the border).
// In the difference arrays (2^-40) that is +beta v at max(x-1, 0) and -beta v at x+1 (if inside)
// of the row, the same along the column.  Global-memory form (global tiles); also accumulates the
// turning point's share of E[TP] and of the border deficit B = sum_v VD_v (4 - deg(v)).
__device__ __forceinline__ void tp_fold_global(const KParams& P, const StepArgs& A, int x, int y, int v,
                                               long long& etp, long long& bdef) {
  if (v == 0) return;
  const long long b = beta_fold(A, v);
  const int X = P.X, Y = P.Y;
  red64(P.dH + (size_t)y * X + max(x - 1, 0), b);
  if (x + 1 <= X - 1) red64(P.dH + (size_t)y * X + x + 1, -b);
  red64(P.dVT + (size_t)x * Y + max(y - 1, 0), b);
  if (y + 1 <= Y - 1) red64(P.dVT + (size_t)x * Y + y + 1, -b);
  etp += v;
  bdef += (long long)v * border_deficit(x, y, X, Y);
}

// Flush of a tile's event window into the global difference arrays.  The window's three fields are
// int32 (2^-24), row-major over the window with row pitch ep >= ww (cell (x, y) at (y - wy0) ep +
// x - wx0): H events at 0, V events at hv, turning points VD at 2 hv; width and pitch are even, so
// pair i of row r is cells 2i, 2i+1 of that row.  Global cell j of a row receives (H_j << 16) + beta (VD_{j+1} - VD_{j-1} + [j = 0] VD_0):
// its wire events and the turning points' +-beta pi windows along the row (tp_fold_global); cell j
// of a column likewise with V and the VD of the cells above / below.  One pass, four predicated
// int64 reductions per pair; cells outside the grid hold no events and receive nothing.  Returns
// the window's share of E[TP] = sum VD and of the border deficit B = sum VD (4 - deg) (2^-24); KG
// derives E[WL] from the folded demand and these two (kg_loss_kernel).
template <int NT, bool EXACT>
__device__ __forceinline__ void flush_window_t(const KParams& P, const StepArgs& A, int wx0, int wy0, int ww, int wh,
                                               int ep, int hv, const int* ev_s, long long& etp, long long& bdef) {
  const int X = P.X, Y = P.Y, tid = threadIdx.x;
  const int hw = ww >> 1, hp = ep >> 1;   // pairs per row: of the window, of the (even) pitch
  // row = floor((i + 1/2) / half width) in fp32 is exact here: the fraction stays >= 1/(2 half)
  // >> the rounding of i < 2^12
  const float inv_hw = 1.f / (float)hw;
  const int2* evH = reinterpret_cast<const int2*>(ev_s);
  const int2* evV = reinterpret_cast<const int2*>(ev_s + hv);
  const int* evD = ev_s + 2 * hv;
  const int2* evD2 = reinterpret_cast<const int2*>(evD);
  const int npair = hw * wh;
  const int bq = (int)A.beta_qi;   // EXACT: beta 2^16 (|beta| < 2^15)
  // windows that reach past the grid's last row / column (their outer cells hold no events but
  // must not be flushed) and windows on the grid border (clipped turning-point windows) take the
  // checked path; the rest (nearly all) need no per-cell test
  const bool plain = wx0 > 0 && wy0 > 0 && wx0 + ww < X && wy0 + wh < Y;
  for (int i = tid; i < npair; i += NT) {
    const int r = (int)(((float)i + 0.5f) * inv_hw), cx = 2 * (i - r * hw);
    const int gx = wx0 + cx, gy = wy0 + r;
    const int pi = r * hp + (cx >> 1);   // the pair in the pitched fields
    const int2 h = evH[pi], v = evV[pi], d = evD2[pi];
    const int dl = cx > 0 ? evD[2 * pi - 1] : 0, dr = cx + 2 < ww ? evD[2 * pi + 2] : 0;
    const int2 du = r > 0 ? evD2[pi - hp] : make_int2(0, 0), dn = r + 1 < wh ? evD2[pi + hp] : make_int2(0, 0);
    if (((h.x | h.y | v.x | v.y | d.x | d.y | dl | dr) | (du.x | du.y | dn.x | dn.y)) == 0) continue;   // nothing to flush
    // turning-point counts are >= 0 and < 2^31 per cell, so these differences fit int32
    int fh0 = d.y - dl, fh1 = dr - d.x, fv0 = dn.x - du.x, fv1 = dn.y - du.y;
    etp += (long long)d.x + d.y;
    const size_t gH = (size_t)gy * X + gx, gV = (size_t)gx * Y + gy;
    long long a0, a1, b0, b1;
    if (EXACT) {
      a0 = (long long)h.x * 65536 + (long long)fh0 * bq;
      a1 = (long long)h.y * 65536 + (long long)fh1 * bq;
      b0 = (long long)v.x * 65536 + (long long)fv0 * bq;
      b1 = (long long)v.y * 65536 + (long long)fv1 * bq;
    } else {
      a0 = ((long long)h.x << kGridShift) + beta_fold(A, fh0);
      a1 = ((long long)h.y << kGridShift) + beta_fold(A, fh1);
      b0 = ((long long)v.x << kGridShift) + beta_fold(A, fv0);
      b1 = ((long long)v.y << kGridShift) + beta_fold(A, fv1);
    }
    if (!plain) {
      // clipped windows of turning points on the first row / column start at edge 0; cells outside
      // the grid receive nothing; border cells have fewer incident edges (B)
      if (gx == 0) a0 += beta_fold<EXACT>(A, d.x);
      if (gy == 0) { b0 += beta_fold<EXACT>(A, d.x); b1 += beta_fold<EXACT>(A, d.y); }
      if (!(gx < X && gy < Y)) { a0 = 0; b0 = 0; }
      if (!(gx + 1 < X && gy < Y)) { a1 = 0; b1 = 0; }
      if (gy < Y) bdef += (long long)d.x * border_deficit(gx, gy, X, Y) + (long long)d.y * border_deficit(gx + 1, gy, X, Y);
    }
    red64p(P.dH + gH, a0);
    red64p(P.dH + gH + 1, a1);
    red64p(P.dVT + gV, b0);
    red64p(P.dVT + gV + Y, b1);
  }
}

template <int NT>
__device__ __forceinline__ void flush_window(const KParams& P, const StepArgs& A, int wx0, int wy0, int ww, int wh,
                                             int ep, int hv, const int* ev_s, long long& etp, long long& bdef) {
  if (A.beta_exact) flush_window_t<NT, true>(P, A, wx0, wy0, ww, wh, ep, hv, ev_s, etp, bdef);
  else flush_window_t<NT, false>(P, A, wx0, wy0, ww, wh, ep, hv, ev_s, etp, bdef);
}

__device__ __forceinline__ long long warp_sum_ll(long long v) {
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) v += __shfl_down_sync(kFull, v, off);
  return v;
}

__device__ __forceinline__ void adam_update(float& w, float& m, float& v, float g, const StepArgs& A) {
  m = fmaf(0.1f, g - m, m);                         // m.lerp_(g, 1 - beta1)
  v = fmaf(0.999f, v, 0.001f * g * g);              // v * beta2 + (1 - beta2) g^2
  // MUFU square root and division: ~1e-7 relative, well inside the 1e-4 bar
  float sq;
#if DGR_ACCURATE
  sq = sqrtf(v);
#else
  asm("sqrt.approx.f32 %0, %1;" : "=f"(sq) : "f"(v));
#endif
  const float denom = sq * A.inv_sqrt_bc2 + 1e-8f;
  w -= A.lr_over_bc1 * FDIV(m, denom);
}

// ------------------------------------------------------------------------------------------
// Grid accessors: the same code runs against the tile's shared-memory window or, for global
// tiles, against the whole grid in HBM.  One base pointer: S_H (row-major) at [0, hv) and
// S_V (column-major) at [hv, 2 hv); the same for the H / V demand-event windows.
// ------------------------------------------------------------------------------------------
struct Win {
  int ox, oy, hs, vs, hv;   // origin; row stride of H (= width); column stride of V (= height); V offset
  __device__ __forceinline__ int h(int x, int y) const { return (y - oy) * hs + (x - ox); }
  __device__ __forceinline__ int v(int x, int y) const { return hv + (x - ox) * vs + (y - oy); }
};

// Orientation-neutral pattern form.  Every pattern is "Z(o, m)": o = 0 lays the first and third
// segments along H rows (straight H, HV, Z-HVH), o = 1 along V columns (straight V, VH, Z-VHV).
// With (p, q) = (x, y) for o = 0 and (y, x) for o = 1, the sub-net runs from (p0, q0) to (p1, q1)
// and the pattern word carries m:
//   seg 1: primary line q0 from p0 to m;     seg 2: secondary line m from q0 to q1;
//   seg 3: primary line q1 from m to p1;     turning points (m, q0) [ntp >= 1], (m, q1) [ntp = 2].
// L shapes have m = p1 (seg 3 empty, one turning point), straight paths m = p1 and q0 = q1, Z
// shapes m strictly between p0 and p1, C-shapes (row f4, Q14b) m outside [p0, p1].  For the Shape
// enum o = shape & 1 and ntp = shape >> 1.  A segment "from a to b" covers the edges
// [min(a,b), max(a,b)) of its line, so its G sum is sgn(b - a) (S[b] - S[a]), S the line's
// exclusive prefix.
__device__ __forceinline__ int isgn(int d) { return (d > 0) - (d < 0); }

// detour length of a C-shape (row f4, reading Q14b): how far x_m / y_m lies outside the span
__device__ __forceinline__ int detour(uint32_t pw, int x0, int y0, int x1, int y1) {
  if (!(pw & kOutside)) return 0;
  const int m = (int)(pw >> 16);
  if ((pw & 7u) == kZHVH) return m < x0 ? x0 - m : m - x1;
  const int ylo = min(y0, y1), yhi = max(y0, y1);
  return m < ylo ? ylo - m : m - yhi;
}

// c_i = a1 WL + a2 sqrt(L) TP + sum over the path's edges of G + beta sum over its turning points
// of the G of the incident edges (Eqs. (9)-(12) chain rule, reading Q3).  Element (a, b) of
// orientation o (H: a = y, b = x; V: a = x, b = y) of the window / grid W is at a * L[o] + b + B[o].
__device__ __forceinline__ double path_cost(const double* S, const Win& W, int X, int Y, uint32_t pw, int x0,
                                            int y0, int x1, int y1, const StepArgs& A) {
  const int o = pw & 1, ntp = (pw >> 1) & 3, m = (int)(pw >> 16);
  const int p0 = o ? y0 : x0, p1 = o ? y1 : x1, q0 = o ? x0 : y0, q1 = o ? x1 : y1;
  const int Lp = o ? W.vs : W.hs, Ls = o ? W.hs : W.vs;
  const int B0 = -(W.oy * W.hs + W.ox), B1 = W.hv - W.ox * W.vs - W.oy;
  const int Bp = o ? B1 : B0, Bs = o ? B0 : B1;
  const int r0 = q0 * Lp + Bp, r1 = q1 * Lp + Bp, sb = m * Ls + Bs;
  const int a0 = r0 + m, a1 = r1 + m, s0 = sb + q0, s1 = sb + q1;
  // each segment's G sum as S[max] - S[min] (a zero-length segment gives 0)
  double c = (S[r0 + max(p0, m)] - S[r0 + min(p0, m)]) + (S[sb + max(q0, q1)] - S[sb + min(q0, q1)]) +
             (S[r1 + max(m, p1)] - S[r1 + min(m, p1)]);
  // turning-point windows: the (clipped) edges left / right and below / above the cell
  const int pmax = (o ? Y : X) - 1, qmax = (o ? X : Y) - 1;
  const int mp = m < pmax, mn = m > 0;
  double tp = 0.0;
  if (ntp >= 1) tp = (S[a0 + mp] - S[a0 - mn]) + (S[s0 + (q0 < qmax)] - S[s0 - (q0 > 0)]);
  if (ntp == 2) tp += (S[a1 + mp] - S[a1 - mn]) + (S[s1 + (q1 < qmax)] - S[s1 - (q1 > 0)]);
  const int wl = abs(m - p0) + abs(p1 - m) + abs(q1 - q0);
  return c + A.beta_d * tp + A.a_wl_d * (double)wl + A.via_d * (double)ntp;
}

// wire length of a candidate in the Z(o, m) form (every shape: straight, L, Z, C)
__device__ __forceinline__ int lane_wl(uint32_t pw, int x0, int y0, int x1, int y1) {
  const int o = pw & 1, m = (int)(pw >> 16);
  const int p0 = o ? y0 : x0, p1 = o ? y1 : x1, q0 = o ? x0 : y0, q1 = o ? x1 : y1;
  return abs(m - p0) + abs(p1 - m) + abs(q1 - q0);
}

__device__ __forceinline__ void red_shared_add(uint32_t saddr, int v) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.s32 p, %1, 0;\n\t@p red.shared.add.s32 [%0], %1;\n\t}" ::"r"(saddr), "r"(v)
               : "memory");
}

// A C-shape lane's own demand events (its corners are not shared with the L / Z collapse):
// emit(field, x, y, value) with field 0 = dH (rows), 1 = dV (columns), 2 = turning points.
template <typename Emit>
__device__ __forceinline__ void c_events(uint32_t pw, int x0, int y0, int x1, int y1, int v, Emit emit) {
  const int m = (int)(pw >> 16);
  const int ylo = min(y0, y1), yhi = max(y0, y1);
  if ((pw & 7u) == kZHVH) {
    emit(0, min(x0, m), y0, v); emit(0, max(x0, m), y0, -v);
    emit(0, min(m, x1), y1, v); emit(0, max(m, x1), y1, -v);
    emit(1, m, ylo, v); emit(1, m, yhi, -v);
    emit(2, m, y0, v); emit(2, m, y1, v);
  } else {
    emit(1, x0, min(y0, m), v); emit(1, x0, max(y0, m), -v);
    emit(1, x1, min(m, y1), v); emit(1, x1, max(m, y1), -v);
    emit(0, x0, m, v); emit(0, x1, m, -v);
    emit(2, x0, m, v); emit(2, x1, m, v);
  }
}


// Lane view built from already-loaded bundle info and pattern word (no memory access).
__device__ __forceinline__ void lane_from(int4 bi, uint32_t pw, const KParams& P, Lane& L) {
  L.lane = threadIdx.x & 31;
  L.pw = pw;
  L.shape = pw & 7u;
  L.valid = L.shape != kPad;
  L.hm = __ballot_sync(kFull, pw & kSubHead);
  L.tm = __ballot_sync(kFull, pw & kTreeHead);
  L.le = kFull >> (31 - L.lane);
  L.head = 31 - __clz(L.hm & L.le);
  const uint32_t rest = L.hm & ~L.le;
  L.end = rest ? (__ffs(rest) - 2) : 31;
  L.gmask = (kFull >> (31 - L.end)) & ~((1u << L.head) - 1u);
  L.sub = bi.y + __popc(L.hm & L.le) - 1;
  L.tree = bi.z + (int)((pw >> kTreeShift) & kTreeMask);
  L.single = (bi.w & kSingleBundle) != 0;
}

// p_i = exp(z_i - m) / sum_k exp(z_k - m) for any shift m (softmax shift invariance): m = the group
// head's z, unless some lane of the warp exceeds its head by more than 64 (exp overflow risk), then
// the exact group maximum.  The head's own term is exp(0) = 1, so the sum is >= 1.
// Lane view of a group-bundle slot from its plan-time lane descriptor (no ballots): head / end lane
// of its group, its sub-net (bundle's first + index), tree; the fields a group lane needs.
__device__ __forceinline__ void lane_from_desc(int4 bi, uint32_t pw, uint32_t ld, Lane& L) {
  L.lane = threadIdx.x & 31;
  L.pw = pw;
  L.shape = pw & 7u;
  L.valid = L.shape != kPad;
  L.head = (int)((ld >> 11) & 31u);
  L.end = (int)((ld >> 16) & 31u);
  L.sub = bi.y + (int)((ld >> 21) & 31u);
  L.tree = bi.z + (int)((pw >> kTreeShift) & kTreeMask);
  L.single = false;
}

__device__ __forceinline__ float softmax_from_noise(const Lane& L, float w, float g, float inv_t) {
  const float z = L.valid ? (w + g) * inv_t : -INFINITY;
  float m = __shfl_sync(kFull, z, L.head);
  if (!DGR_HEAD_SOFTMAX || __any_sync(kFull, z - m > 64.f)) {
    m = seg_reduce(z, L.lane, L.end, Max());
    m = __shfl_sync(kFull, m, L.head);
  }
  const float e = L.valid ? FEXP(z - m) : 0.f;
  float s = seg_reduce(e, L.lane, L.end, Sum());
  s = __shfl_sync(kFull, s, L.head);
  return L.valid ? FDIV(e, s) : 0.f;
}

// ------------------------------------------------------------------------------------------
// The tile kernel.  Shared memory (dynamic), region A is reused between the two halves:
//   A, reverse:  S_s   double[2 kWinMax]          S window: H part, then V part
//   A, forward:  ev_s  int[3 kWinMax]             demand-event window dH | dV | VD, 2^-24 fixed point
//                g_s   float[kWarps][kWarpCand]   Gumbel noise of each warp's candidates
//   wst    float[kMaxBundles * 32]    new logits of the tile (reverse -> forward)
//   dq_s   long long[kTreeMax]        dq_j in 2^-32 fixed point
//   q_s    float[kTreeMax]            q_j (iteration k in the reverse, k_next in the forward)
// Each warp owns a contiguous range of the tile's bundles, so its candidates are contiguous.
// ------------------------------------------------------------------------------------------
constexpr int kWarps = kTileThreads / 32;
constexpr int kWarpBundles = (kMaxBundles + kWarps - 1) / kWarps;
constexpr int kWarpCand = kWarpBundles * 32;
constexpr size_t kRegionA = (2 * sizeof(double) * kWinMax > 3 * sizeof(int) * kWinMax + sizeof(float) * kWarps * kWarpCand)
                               ? 2 * sizeof(double) * kWinMax
                               : 3 * sizeof(int) * kWinMax + sizeof(float) * kWarps * kWarpCand;
constexpr size_t kSmemBytes = kRegionA + sizeof(float) * kMaxBundles * 32 + sizeof(long long) * kTreeMax +
                              sizeof(float) * kTreeMax + 2 * sizeof(long long);

template <bool GLOBAL>
__device__ __forceinline__ void reverse_warp(const KParams& P, const StepArgs& A, const TileDesc& T, int bw0,
                                             int bw1, const double* S, const Win& W, long long* dq_s,
                                             const float* q_s, float* wst) {
  const int lane = threadIdx.x & 31;
  // software pipeline: bundle b computes while b+1's operands (incl. its sub-net endpoints, which
  // depend on b+1's ballots) and b+2's bundle info / pattern word are in flight
  size_t slot = (size_t)bw0 * 32 + lane;
  Lane L;
  lane_from(__ldg(&P.binfo[bw0]), __ldg(&P.pword[slot]), P, L);
  short4 e = L.valid ? __ldg(&P.sxy[L.sub]) : make_short4(0, 0, 0, 0);
  float w = P.wp[slot], m = P.mv[slot].x, v = P.mv[slot].y, p = P.pp[slot];
  int4 bi1 = make_int4(0, 0, 0, 0);
  uint32_t pw1 = kPad | kSubHead;
  if (bw0 + 1 < bw1) { bi1 = __ldg(&P.binfo[bw0 + 1]); pw1 = __ldg(&P.pword[slot + 32]); }
  for (int b = bw0; b < bw1; ++b) {
    Lane Ln = L;
    short4 en = e;
    float wn = w, mn = m, vn = v, pn = p;
    if (b + 1 < bw1) {
      lane_from(bi1, pw1, P, Ln);
      if (Ln.valid) en = __ldg(&P.sxy[Ln.sub]);
      wn = P.wp[slot + 32]; mn = P.mv[slot + 32].x; vn = P.mv[slot + 32].y; pn = P.pp[slot + 32];
      if (b + 2 < bw1) { bi1 = __ldg(&P.binfo[b + 2]); pw1 = __ldg(&P.pword[slot + 64]); }
    }
    const float q = L.valid ? q_s[L.tree - T.tree0] : 0.f;
    const double c = L.valid ? path_cost(S, W, P.X, P.Y, L.pw, e.x, e.y, e.z, e.w, A) : 0.0;
    // softmax backward dw_i = (p_i/t)(dp_i - sum_k p_k dp_k / sum_k p_k): differences to the group
    // head's dp are formed in fp64 and reduced in fp32, so neither the magnitude of c nor
    // sum_k p_k != 1 (rounding) leaks into dw.
    // exactly the arithmetic of process_tile (pipelined tiles), so that a net gives bit-identical
    // results whichever kind of tile it lands in (tile composition depends on the rank count):
    if (L.single) {
      // singleton bundle (lone straight sub-nets, p = 1): tree-run sums of c into dq; no Adam (the
      // logit of a lone straight candidate never changes)
      const uint32_t th = __ballot_sync(kFull, (L.pw & kTreeHead) || !L.valid) | 1u;
      const uint32_t trest = th & ~L.le;
      const int tend = trest ? (__ffs(trest) - 2) : 31;
      const long long pc = seg_reduce(L.valid ? __double2ll_rn(c * kDqScale) : 0ll, L.lane, tend, Sum());
      if (L.valid && ((th >> L.lane) & 1u))
        atomicAdd(reinterpret_cast<unsigned long long*>(&dq_s[L.tree - T.tree0]), static_cast<unsigned long long>(pc));
    } else {
      // softmax backward over the sub-net with dd = c - c_head (fp64 difference, then fp32):
      // dw_i = (p_i / t) q (dd_i - sum_k p_k dd_k); the head adds c_head + sum_k p_k dd_k to dq
      const double ch = __shfl_sync(kFull, c, L.head);
      const float dd = (float)(c - ch);
      float sa = seg_reduce(p * dd, L.lane, L.end, Sum());
      sa = __shfl_sync(kFull, sa, L.head);
      const float dw = L.valid ? p * A.inv_t * q * (dd - sa) : 0.f;
      if (L.valid && L.lane == L.head)
        atomicAdd(reinterpret_cast<unsigned long long*>(&dq_s[L.tree - T.tree0]),
                  static_cast<unsigned long long>(__double2ll_rn((c + (double)sa) * kDqScale)));
      if (L.valid) {
        adam_update(w, m, v, dw, A);
        P.wp[slot] = w;
        P.mv[slot] = make_float2(m, v);
      }
    }
    wst[(b - T.b0) * 32 + lane] = w;
    L = Ln; e = en; w = wn; m = mn; v = vn; p = pn;
    slot += 32;
  }
}

// Forward events of one lane.  For a canonical sub-net (x0 < x1), s = sgn(y1 - y0), the +-pi events
// of all its candidates collapse onto 4 corner G-cells plus 2 cells per Z candidate:
//   (x0,y0): dH += A+Hs, dV += s(B+Vs)        (x1,y0): dH -= A, dV += sA, VD += A      [HV lane]
//   (x0,y1): dH += B, dV -= sB, VD += B       (x1,y1): dH -= B+Hs, dV -= s(A+Vs)       [VH lane]
//   Z-HVH(xm): (xm,y0): -pi, +s pi, +pi   (xm,y1): +pi, -s pi, +pi        [dH, dV, VD]
//   Z-VHV(ym): (x0,ym): +pi, -s pi, +pi   (x1,ym): -pi, +s pi, +pi
// with A = pi_HV, B = pi_VH, Hs = sum pi over Z-HVH, Vs = sum pi over Z-VHV.  dH is the difference
// array of the H wire demand along rows, dV along columns, VD the turning points.  Written as
// 0/1-flag arithmetic so the warp never diverges on the pattern.
// Event window of a tile (row-major fields: H at 0, V at hv, turning points at 2 hv)
struct EWin {
  int ox, oy, w, hv;
  __device__ __forceinline__ int h(int x, int y) const { return (y - oy) * w + (x - ox); }
  __device__ __forceinline__ int v(int x, int y) const { return hv + (y - oy) * w + (x - ox); }
  __device__ __forceinline__ int d(int x, int y) const { return 2 * hv + (y - oy) * w + (x - ox); }
};

template <bool GLOBAL>
__device__ __forceinline__ void forward_warp(const KParams& P, const StepArgs& A, const TileDesc& T, int bw0,
                                             int bw1, bool have_w, const float* wst, const float* q_s, const float* gt,
                                             const EWin& W, int* ev_s, long long& etp, long long& bdef) {
  const int lane = threadIdx.x & 31;
  const int4 bfirst = __ldg(&P.binfo[bw0]);
  const uint32_t ev_base = (uint32_t)__cvta_generic_to_shared(ev_s);
  size_t slot = (size_t)bw0 * 32 + lane;
  Lane L;
  lane_from(bfirst, __ldg(&P.pword[slot]), P, L);
  short4 e = L.valid ? __ldg(&P.sxy[L.sub]) : make_short4(0, 0, 0, 0);
  int4 bi1 = make_int4(0, 0, 0, 0);
  uint32_t pw1 = kPad | kSubHead;
  if (bw0 + 1 < bw1) { bi1 = __ldg(&P.binfo[bw0 + 1]); pw1 = __ldg(&P.pword[slot + 32]); }
  for (int b = bw0; b < bw1; ++b) {
    Lane Ln = L;
    short4 en = e;
    if (b + 1 < bw1) {
      lane_from(bi1, pw1, P, Ln);
      if (Ln.valid) en = __ldg(&P.sxy[Ln.sub]);
      if (b + 2 < bw1) { bi1 = __ldg(&P.binfo[b + 2]); pw1 = __ldg(&P.pword[slot + 64]); }
    }
    const float w = have_w ? wst[(b - T.b0) * 32 + lane] : P.wp[slot];
    const float g = (L.valid && !L.single) ? gumbel_word(__float_as_uint(gt[__ldg(&P.ldesc[slot]) & 0x7FFu])) : 0.f;
    const float p = softmax_from_noise(L, w, g, A.inv_t);
    P.pp[slot] = p;
    const float q = L.valid ? q_s[L.tree - T.tree0] : 0.f;
    const int vq = L.valid ? __float2int_rn(q * p * kFixScale) : 0;   // pi in 2^-24 fixed point
    int sc = vq;                                                       // inclusive scan within the group
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
      const int o = __shfl_up_sync(kFull, sc, off);
      if (L.lane - off >= L.head) sc += o;
    }
    const bool outside = (L.pw & kOutside) != 0;   // C-shape lanes: own events, outside the collapse
    const int nh = __popc(__ballot_sync(kFull, L.shape == kZHVH && !outside) & L.gmask);
    const int nv = __popc(__ballot_sync(kFull, L.shape == kZVHV && !outside) & L.gmask);
    const int h1 = min(L.head + 1, 31), h2 = min(L.head + 1 + nh, 31), h3 = min(L.head + 1 + nh + nv, 31);
    const int a = __shfl_sync(kFull, vq, L.head);
    const int bb = __shfl_sync(kFull, vq, h1);
    const int S1 = __shfl_sync(kFull, sc, h1);
    const int S2 = __shfl_sync(kFull, sc, h2);
    const int S3 = __shfl_sync(kFull, sc, h3);
    const int x0 = e.x, y0 = e.y, x1 = e.z, y1 = e.w;
    const int s = (y1 > y0) ? 1 : -1;
    const int hs = S2 - S1, vs = S3 - S2, v = vq;
    const int mm = (int)(L.pw >> 16);
    const int fSH = L.shape == kStraightH, fSV = L.shape == kStraightV, fHV = L.shape == kHV;
    const int fVH = L.shape == kVH, fZH = L.shape == kZHVH && !outside, fZV = L.shape == kZVHV && !outside;
    const int fZ = fZH + fZV;
    const int xa = x0 + fZH * (mm - x0);
    const int ya = y0 + fVH * (y1 - y0) + fZV * (mm - y0);
    const int xb = x1 + fSV * (x0 - x1) + fZH * (mm - x1);
    const int yb = y1 + (fSH + fHV) * (y0 - y1) + fZV * (mm - y1);
    const int ah = fSH * v + fHV * (a + hs) + fVH * bb + (fZV - fZH) * v;
    const int av = fSV * v + s * (fHV * (bb + vs) - fVH * bb + (fZH - fZV) * v);
    const int ad = fVH * bb + fZ * v;
    const int bh = -fSH * v - fHV * a - fVH * (bb + hs) + (fZH - fZV) * v;
    const int bv = -fSV * v + s * (fHV * a - fVH * (a + vs) + (fZV - fZH) * v);
    const int bd = fHV * a + fZ * v;
    if (L.valid) {
      if (GLOBAL) {
        const int X = P.X, Y = P.Y;
        const long long sh = 1ll << kGridShift;
        red64(P.dH + (size_t)ya * X + xa, ah * sh); red64(P.dVT + (size_t)xa * Y + ya, av * sh);
        tp_fold_global(P, A, xa, ya, ad, etp, bdef);
        red64(P.dH + (size_t)yb * X + xb, bh * sh); red64(P.dVT + (size_t)xb * Y + yb, bv * sh);
        tp_fold_global(P, A, xb, yb, bd, etp, bdef);
      }
      if (outside) {
        if (GLOBAL) {
          const int X = P.X, Y = P.Y;
          c_events(L.pw, x0, y0, x1, y1, vq, [&](int fld, int x, int y, int val) {
            if (fld == 2) tp_fold_global(P, A, x, y, val, etp, bdef);
            else red64(fld == 0 ? P.dH + (size_t)y * X + x : P.dVT + (size_t)x * Y + y, (long long)val << kGridShift);
          });
        } else {
          c_events(L.pw, x0, y0, x1, y1, vq, [&](int fld, int x, int y, int val) {
            red_shared_add(ev_base + 4u * (fld == 0 ? W.h(x, y) : fld == 1 ? W.v(x, y) : W.d(x, y)), val);
          });
        }
      }
    }
    if (!GLOBAL) {
      red_shared_add(ev_base + 4u * W.h(xa, ya), ah);
      red_shared_add(ev_base + 4u * W.v(xa, ya), av);
      red_shared_add(ev_base + 4u * W.d(xa, ya), ad);
      red_shared_add(ev_base + 4u * W.h(xb, yb), bh);
      red_shared_add(ev_base + 4u * W.v(xb, yb), bv);
      red_shared_add(ev_base + 4u * W.d(xb, yb), bd);
    }
    L = Ln; e = en;
    slot += 32;
  }

}

// The tile body for "global" tiles (nets spanning more than a window, or too many events on a
// window cell): operands straight from global memory, no TMA stage.  Run by the first CTAs of the
// tile_bulk launch (so these long tiles start first and overlap the pipelined ones) or by
// tile_kernel (persistent driver).
template <bool REV, bool FWD>
__device__ __forceinline__ void slow_tile(const KParams& P, const StepArgs& A, const TileDesc T, unsigned char* smem) {
  double* S_s = reinterpret_cast<double*>(smem);                 // region A (reverse)
  int* ev_s = reinterpret_cast<int*>(smem);                      // region A (forward)
  float* g_all = reinterpret_cast<float*>(ev_s + 3 * kWinMax);   // region A (forward)
  float* wst = reinterpret_cast<float*>(smem + kRegionA);
  long long* dq_s = reinterpret_cast<long long*>(wst + kMaxBundles * 32);
  float* q_s = reinterpret_cast<float*>(dq_s + kTreeMax);

  const int tid = threadIdx.x, warp = tid >> 5;
  const int ncell = T.ww * T.wh;
  const Win Wg{0, 0, P.XP, P.YP, (int)(P.SVT - P.SH)};
  const Win Ws{T.wx0, T.wy0, T.ww, T.wh, ncell};
  // this warp's contiguous bundle range
  const int per = (T.nb + kWarps - 1) / kWarps;
  const int bw0 = T.b0 + min(warp * per, T.nb), bw1 = T.b0 + min((warp + 1) * per, T.nb);

  // ---------------- reverse of iteration k ----------------
  if (REV && !(KO(64))) {
    if (!T.global) {
      const int lane = tid & 31;
      for (int yi = warp; yi < T.wh; yi += kWarps) {
        const double* src = P.SH + (size_t)(T.wy0 + yi) * P.XP + T.wx0;
        for (int xi = lane; xi < T.ww; xi += 32) S_s[yi * T.ww + xi] = src[xi];
      }
      for (int xi = warp; xi < T.ww; xi += kWarps) {
        const double* src = P.SVT + (size_t)(T.wx0 + xi) * P.YP + T.wy0;
        for (int yi = lane; yi < T.wh; yi += 32) S_s[ncell + xi * T.wh + yi] = src[yi];
      }
    }
    for (int i = tid; i < T.ntree; i += kTileThreads) { dq_s[i] = 0; q_s[i] = P.q[T.tree0 + i]; }
    __syncthreads();
    if (bw0 < bw1) {
      if (T.global) reverse_warp<true>(P, A, T, bw0, bw1, P.SH, Wg, dq_s, q_s, wst);
      else reverse_warp<false>(P, A, T, bw0, bw1, S_s, Ws, dq_s, q_s, wst);
    }
    __syncthreads();
  }

  // ---------------- tree level ----------------
  for (int n = tid; n < T.nnet; n += kTileThreads) {
    const int net = T.net0 + n;
    const int a = P.net_tree_off[net], b = P.net_tree_off[net + 1];
    if (REV) {
      // du_j = (q_j/t)(dq_j - sum_l q_l dq_l / sum_l q_l); Adam on w_tree (iteration k)
      double sq = 0.0, sw = 0.0;
      for (int j = a; j < b; ++j) {
        const double qj = (double)q_s[j - T.tree0];
        sq += qj * ((double)dq_s[j - T.tree0] * kDqInv);
        sw += qj;
      }
      sq /= sw;
      for (int j = a; j < b; ++j) {
        const double du = (b - a == 1) ? 0.0
                                       : (double)q_s[j - T.tree0] * (double)A.inv_t * ((double)dq_s[j - T.tree0] * kDqInv - sq);
        float w = P.wt[j], m = P.mt[j], v = P.vt[j];
        adam_update(w, m, v, (float)du, A);
        P.wt[j] = w; P.mt[j] = m; P.vt[j] = v;
      }
    }
    if (FWD) {
      // q_j = softmax over the net's trees of (w_j + g_j)/t, iteration k_next (stream 1)
      if (b - a == 1) {
        q_s[a - T.tree0] = 1.f;
        P.q[a] = 1.f;
      } else {
        float zmax = -INFINITY;
        for (int j = a; j < b; ++j) {
          const float z = (P.wt[j] + gumbel(P.seed, (uint64_t)(P.tree_base + P.net_gtree[net] + (j - a)), (uint32_t)A.k_next, 1u)) * A.inv_t;
          q_s[j - T.tree0] = z;
          zmax = fmaxf(zmax, z);
        }
        float sum = 0.f;   // the normalisation of process_tile, operation for operation
        for (int j = a; j < b; ++j) sum += FEXP(q_s[j - T.tree0] - zmax);
        for (int j = a; j < b; ++j) {
          const float q = FEXP(q_s[j - T.tree0] - zmax) / sum;
          q_s[j - T.tree0] = q;
          P.q[j] = q;
        }
      }
    }
  }

  // ---------------- forward of iteration k_next ----------------
  if (FWD) {
    if (!T.global) {
      int4* z = reinterpret_cast<int4*>(ev_s);
      for (int i = tid; i < (3 * ncell + 3) / 4; i += kTileThreads) z[i] = make_int4(0, 0, 0, 0);
    }
    if (T.nbg > 0) tile_noise<kTileThreads>(P, T, (uint32_t)A.k_next, g_all);   // path noise by tile noise offset
    __syncthreads();
    long long etp = 0, bdef = 0;
    const EWin Ew{T.wx0, T.wy0, T.ww, ncell};
    if (bw0 < bw1) {
      if (T.global) forward_warp<true>(P, A, T, bw0, bw1, REV, wst, q_s, g_all, Ew, ev_s, etp, bdef);
      else forward_warp<false>(P, A, T, bw0, bw1, REV, wst, q_s, g_all, Ew, ev_s, etp, bdef);
    }
    __syncthreads();
    if (!T.global) flush_window<kTileThreads>(P, A, T.wx0, T.wy0, T.ww, T.wh, T.ww, ncell, ev_s, etp, bdef);
    etp = warp_sum_ll(etp);
    bdef = warp_sum_ll(bdef);
    if ((tid & 31) == 0 && (etp | bdef)) {   // exact integers: any order gives the same sums
      atomicAdd(reinterpret_cast<unsigned long long*>(P.acc), (unsigned long long)etp);
      atomicAdd(reinterpret_cast<unsigned long long*>(P.acc + 1), (unsigned long long)bdef);
    }
  }
}


// ------------------------------------------------------------------------------------------
// Persistent, TMA-pipelined tile kernel (the hot loop).  One CTA per SM walks its tiles
// (blockIdx.x, +gridDim.x, ...).  While tile i is processed out of shared-memory stage s, the
// bulk-copy engine (cp.async.bulk, completion on an mbarrier) fills stage s^1 with tile i+1's
// operands: pattern words, w, m, v, p of its bundles, bundle info, sub-net endpoints, net->tree
// offsets, tree state, and the tile's S window (one bulk copy per window row of S_H and per
// window column of S_V).  Updated w, m, v, p go back with bulk stores; demand events are
// accumulated in a shared-memory window and flushed with int64 reductions.
// ------------------------------------------------------------------------------------------
constexpr int kPSlots = kTargetBundles * 32;                // 1024
constexpr int kPSubMax = kPipeSubs + 2;                     // + alignment slack
constexpr int kPTreeMax = kPipeTrees + 4;
constexpr int kPNetMax = kPipeTrees + 8;

// The stage keeps what several phases share: pattern words and logits of the tile's slots, bundle
// info, sub-net endpoints, net->tree offsets, the multi-tree net list, tree logits and q, and the S
// window.  Adam moments and the stored p of the paths, and m, v of the trees, are read / written
// directly (each warp its bundle's 128-byte rows), so the stage fits 5 CTAs per SM.
constexpr int kPMnMax = 0;   // (the net level's tree lanes are read straight from mnets, not staged)
struct StageLayout {
  static constexpr size_t pw = 0;
  static constexpr size_t w = pw + 4 * 32 * kTileBundles;
  static constexpr size_t bi = w + 4 * kPSlots;
  static constexpr size_t sxy = bi + 16 * kTileBundles;
  static constexpr size_t nto = sxy + 8 * kPSubMax;
  static constexpr size_t mn = (nto + 4 * kPNetMax + 15) / 16 * 16;
  static constexpr size_t q = (mn + 4 * kPMnMax + 15) / 16 * 16;
  static constexpr size_t wt = q + 4 * kPTreeMax;
  static constexpr size_t S = (wt + 4 * kPTreeMax + 127) / 128 * 128;
  static constexpr size_t bytes = S + 2 * 8 * (kWinMax + kWinPad);
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n\tWAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, %2;\n\t"
      "@!P1 bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)), "r"(parity), "r"(1000000u) : "memory");   // suspend, don't spin
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src)), "r"(bytes)
               : "memory");
}
// L2 eviction policy for data streamed once per iteration (slot state, pattern words, per-bundle
// and per-sub-net records): evict first, so the S prefix sums (re-read by neighbouring tiles) and the
// demand grids (int64 reductions from every tile) stay resident in L2.
#ifndef DGR_L2_HINTS
#define DGR_L2_HINTS 0
#endif
__device__ __forceinline__ uint64_t policy_stream() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void bulk_g2s_stream(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint64_t pol) {
  if (!DGR_L2_HINTS) { bulk_g2s(dst, src, bytes, bar); return; }
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
               ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
               : "memory");
}
__device__ __forceinline__ void bulk_s2g_stream(void* dst, const void* src, uint32_t bytes, uint64_t pol) {
  if (!DGR_L2_HINTS) { bulk_s2g(dst, src, bytes); return; }
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(dst), "r"(smem_u32(src)),
               "r"(bytes), "l"(pol)
               : "memory");
}
__device__ __forceinline__ float ld_stream(const float* p, uint64_t pol) {
  if (!DGR_L2_HINTS) return *p;
  float v;
  asm volatile("ld.global.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ float2 ld_stream2(const float2* p, uint64_t pol) {
  if (!DGR_L2_HINTS) return *p;
  float2 v;
  asm volatile("ld.global.L2::cache_hint.v2.f32 {%0, %1}, [%2], %3;" : "=f"(v.x), "=f"(v.y) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ void st_stream(float* p, float v, uint64_t pol) {
  if (!DGR_L2_HINTS) { *p = v; return; }
  asm volatile("st.global.L2::cache_hint.f32 [%0], %1, %2;" ::"l"(p), "f"(v), "l"(pol) : "memory");
}
__device__ __forceinline__ void st_stream2(float2* p, float2 v, uint64_t pol) {
  if (!DGR_L2_HINTS) { *p = v; return; }
  asm volatile("st.global.L2::cache_hint.v2.f32 [%0], {%1, %2}, %3;" ::"l"(p), "f"(v.x), "f"(v.y), "l"(pol) : "memory");
}
// Programmatic dependent launch: KBF and KG are launched with programmatic stream serialization,
// so the next kernel's CTAs are scheduled into the slots the previous kernel's last wave leaves
// free; each waits here (griddepcontrol.wait: the previous grid has completed and its writes are
// visible) before it touches anything that grid writes.
__device__ __forceinline__ void griddep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void griddep_launch() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

__device__ __forceinline__ void prefetch_l2(const void* src, uint32_t bytes) {
  if (bytes) asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(src), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

struct Stage {
  uint32_t* pw; float* w;
  int4* bi; short4* sxy; int *nto, *mn; float *q, *wt; double* S;
  __device__ __forceinline__ explicit Stage(unsigned char* base) {
    pw = reinterpret_cast<uint32_t*>(base + StageLayout::pw);
    w = reinterpret_cast<float*>(base + StageLayout::w);
    bi = reinterpret_cast<int4*>(base + StageLayout::bi);
    sxy = reinterpret_cast<short4*>(base + StageLayout::sxy);
    nto = reinterpret_cast<int*>(base + StageLayout::nto);
    mn = reinterpret_cast<int*>(base + StageLayout::mn);
    q = reinterpret_cast<float*>(base + StageLayout::q);
    wt = reinterpret_cast<float*>(base + StageLayout::wt);
    S = reinterpret_cast<double*>(base + StageLayout::S);
  }
};

// aligned element ranges of a tile's sub-nets / nets / multi-tree nets / trees (16-byte bulk
// granularity)
__device__ __forceinline__ void tile_ranges(const TileDesc& T, int& s_lo, int& s_hi, int& n_lo, int& n_hi, int& t_lo, int& t_hi) {
  s_lo = T.sub0 & ~1; s_hi = (T.sub0 + T.nsub + 1) & ~1;
  n_lo = T.net0 & ~3; n_hi = (T.net0 + T.nnet + 1 + 3) & ~3;
  t_lo = T.tree0 & ~3; t_hi = (T.tree0 + T.ntree + 3) & ~3;
}

// warp 0 issues the bulk copies of tile T into stage `st`, completing on `bar`
__device__ __forceinline__ void tma_2d(void* dst, const void* tmap, int c0, int c1, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          smem_u32(dst)),
      "l"(tmap), "r"(c0), "r"(c1), "r"(smem_u32(bar))
      : "memory");
}

template <bool REV>
__device__ __forceinline__ void issue_tile_loads(const KParams& P, const TileDesc& T, unsigned char* st, uint64_t* bar,
                                                 bool window = true) {
  const int lane = threadIdx.x & 31;
  Stage S(st);
  int s_lo, s_hi, n_lo, n_hi, t_lo, t_hi;
  tile_ranges(T, s_lo, s_hi, n_lo, n_hi, t_lo, t_hi);
  const uint32_t slot_bytes = (uint32_t)T.nb * 128u, gslot_bytes = (uint32_t)T.nbg * 128u;
  const bool sw = REV && window && !(KO(32));   // knock-out 32: no S window (timing only)
  const uint32_t nrow = sw ? (uint32_t)T.wh : 0u, ncol = sw ? (uint32_t)T.ww : 0u;
  // REV && !window && tmap >= 0: the S window by two 2-D tensor copies (H field, V field)
  const bool tw = REV && !window && T.tmap >= 0 && !(KO(32));
  const uint32_t bytes = slot_bytes + gslot_bytes + 16u * T.nb + 8u * (s_hi - s_lo) + 4u * (n_hi - n_lo) +
                         8u * (t_hi - t_lo) + 8u * (nrow * T.ww + ncol * T.wh) +
                         (tw ? 8u * (uint32_t)(T.wh * win_pitch(T.ww) + T.ww * win_pitch(T.wh)) : 0u);
  if (lane == 0) mbar_expect_tx(bar, bytes);
  __syncwarp();
  const size_t s0 = (size_t)T.b0 * 32;
  const uint64_t pol = policy_stream();
  if (tw && lane == 8) {
    const unsigned char* tm = P.tmaps + 256 * (size_t)T.tmap;
    tma_2d(S.S, tm, T.wx0, T.wy0, bar);
    tma_2d(S.S + win_s_hv(T.ww, T.wh), tm + 128, T.wy0, T.wx0, bar);
  }
  // work items: 0..7 the 1-D arrays, then window rows, then window columns
  const int nitems = 8 + (int)nrow + (int)ncol;
  for (int it = lane; it < nitems; it += 32) {
    if (it < 8) {
      switch (it) {
        case 0: bulk_g2s_stream(S.pw, P.pword + s0, slot_bytes, bar, pol); break;
        case 1: if (gslot_bytes) bulk_g2s_stream(S.w, P.wp + s0, gslot_bytes, bar, pol); break;
        case 2: bulk_g2s_stream(S.bi, P.binfo + T.b0, 16u * T.nb, bar, pol); break;
        case 3: bulk_g2s_stream(S.sxy, P.sxy + s_lo, 8u * (s_hi - s_lo), bar, pol); break;
        case 4: bulk_g2s_stream(S.nto, P.net_tree_off + n_lo, 4u * (n_hi - n_lo), bar, pol); break;
        case 5: break;
        case 6: bulk_g2s(S.wt, P.wt + t_lo, 4u * (t_hi - t_lo), bar); break;
        default: bulk_g2s(S.q, P.q + t_lo, 4u * (t_hi - t_lo), bar); break;   // also a lone tree's q = 1
      }
    } else if (it < 8 + (int)nrow) {
      const int yi = it - 8;
      bulk_g2s(S.S + (size_t)yi * win_pitch(T.ww), P.SH + (size_t)(T.wy0 + yi) * P.XP + T.wx0, 8u * T.ww, bar);
    } else {
      const int xi = it - 8 - (int)nrow;
      bulk_g2s(S.S + win_s_hv(T.ww, T.wh) + (size_t)xi * win_pitch(T.wh), P.SVT + (size_t)(T.wx0 + xi) * P.YP + T.wy0, 8u * T.wh, bar);
    }
  }
}

// The same stage filled by all threads with 16-byte cp.async copies (LSU path, no registers):
// each warp copies one of the eight 1-D arrays, then all threads the S window rows / columns.
// Measured per tile (scratch/tprof.py): the ~90 bulk copies of a tile queue behind those of the
// other resident tiles in the SM's bulk-copy engine (12,000 cycles from issue to arrival).
__device__ __forceinline__ void cp16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_copy(void* dst, const void* src, uint32_t bytes, int lane) {
  char* d = reinterpret_cast<char*>(dst);
  const char* g = reinterpret_cast<const char*>(src);
  for (uint32_t o = 16u * lane; o < bytes; o += 512u) cp16(d + o, g + o);
}
template <bool REV, int NT>
__device__ __forceinline__ void lsu_tile_loads(const KParams& P, const TileDesc& T, unsigned char* st,
                                               bool arrays = true) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  Stage S(st);
  int s_lo, s_hi, n_lo, n_hi, t_lo, t_hi;
  tile_ranges(T, s_lo, s_hi, n_lo, n_hi, t_lo, t_hi);
  const size_t s0 = (size_t)T.b0 * 32;
  if (arrays) switch (warp & 7) {
    case 0: cp_copy(S.pw, P.pword + s0, (uint32_t)T.nb * 128u, lane); break;
    case 1: cp_copy(S.w, P.wp + s0, (uint32_t)T.nbg * 128u, lane); break;
    case 2: cp_copy(S.bi, P.binfo + T.b0, 16u * T.nb, lane); break;
    case 3: cp_copy(S.sxy, P.sxy + s_lo, 8u * (s_hi - s_lo), lane); break;
    case 4: cp_copy(S.nto, P.net_tree_off + n_lo, 4u * (n_hi - n_lo), lane); break;
    case 5: break;
    case 6: cp_copy(S.wt, P.wt + t_lo, 4u * (t_hi - t_lo), lane); break;
    default: cp_copy(S.q, P.q + t_lo, 4u * (t_hi - t_lo), lane); break;
  }
  if (REV && !(KO(32)) && !(arrays == false && T.tmap >= 0)) {
    // S_H window rows (ww doubles = ww/2 chunks each), then S_V window columns (wh/2 chunks each);
    // row = floor((i + 1/2) / half) in fp32 is exact for i < 2^12 (see the flush)
    const int hw = T.ww >> 1, hh = T.wh >> 1, n = hw * T.wh;
    const float inv_hw = 1.f / (float)hw, inv_hh = 1.f / (float)hh;
    for (int i = tid; i < n; i += NT) {
      const int r = (int)(((float)i + 0.5f) * inv_hw), c = i - r * hw;
      cp16(S.S + (size_t)r * win_pitch(T.ww) + 2 * c, P.SH + (size_t)(T.wy0 + r) * P.XP + T.wx0 + 2 * c);
    }
    double* SV = S.S + win_s_hv(T.ww, T.wh);
    for (int i = tid; i < n; i += NT) {
      const int r = (int)(((float)i + 0.5f) * inv_hh), c = i - r * hh;
      cp16(SV + (size_t)r * win_pitch(T.wh) + 2 * c, P.SVT + (size_t)(T.wx0 + r) * P.YP + T.wy0 + 2 * c);
    }
  }
  asm volatile("cp.async.commit_group;" ::: "memory");
}

// L2 prefetch of what a tile reads directly (not through the stage): the group slots' Adam moments
// and stored p, the trees' Adam moments; issued next to the stage's bulk copies, so the direct loads
// of the reverse and net-level phases hit L2.
__device__ __forceinline__ void prefetch_tile(const KParams& P, const TileDesc& T, bool slots = true) {
  const int lane = threadIdx.x & 31;
  const size_t s0 = (size_t)T.b0 * 32;
  const int t_lo = T.tree0 & ~3, t_hi = (T.tree0 + T.ntree + 3) & ~3;
  const uint32_t gs = slots ? (uint32_t)T.nbg * 32u : 0u;
  switch (lane) {
    case 0: if (gs) prefetch_l2(P.mv + s0, 8u * gs); break;
    case 1: if (gs) prefetch_l2(P.pp + s0, 4u * gs); break;
    case 2: prefetch_l2(P.mt + t_lo, 4u * (t_hi - t_lo)); break;
    case 3: prefetch_l2(P.vt + t_lo, 4u * (t_hi - t_lo)); break;
    default: break;
  }
}

// One tile, all operands in shared memory (stage St).  ev_s / gp may alias St.S (they are only
// touched after the reverse half is done with it).  Ends with the slot state written back by bulk
// stores (issued by thread 0, committed) and the demand window flushed.
// Bundles go to warps round-robin; lb < T.nbg are group bundles, the rest singleton bundles (lone
// straight sub-nets: p = 1, no noise, no softmax, no Adam, no slot state).
// Phase timing (DGR_DEBUG_SKIP bit 256, diagnostics only): per pipelined tile, SM clock at
// [start, stage arrived, reverse done, net level done, forward done, end], SM id, global timer.
constexpr int kProfTiles = 16384;
__device__ long long g_tile_prof[kProfTiles * 8];
__device__ __forceinline__ void stamp(const KParams& P, int tile, int k) {
  if ((KO(256)) && threadIdx.x == 0 && tile < kProfTiles) g_tile_prof[tile * 8 + k] = clock64();
}
constexpr size_t kGpOffset = 3 * 4 * (kWinMax + kWinPad);   // tile path noise, after the event window in St.S
template <bool REV, bool FWD, int NT>
__device__ __forceinline__ void process_tile(const KParams& P, const StepArgs& A, const TileDesc& T, Stage St,
                                             int* ev_s, float* gp, int* dq3, uint32_t ld_first, uint32_t mte,
                                             const uint32_t* twd) {
  // dq3[0..3 ntree) arrives zeroed (the caller clears it before its first barrier)
  constexpr int NW = NT / 32;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int X = P.X, Y = P.Y;
  int s_lo, s_hi, n_lo, n_hi, t_lo, t_hi;
  tile_ranges(T, s_lo, s_hi, n_lo, n_hi, t_lo, t_hi);
  const uint64_t pol = policy_stream();   // L2 evict-first for the streamed slot state
  // S window: H rows of pitch win_pitch(ww), V columns of pitch win_pitch(wh) from win_s_hv;
  // event window: row-major fields of pitch ep, hv apart (128-byte aligned)
  const Win W{T.wx0, T.wy0, win_pitch(T.ww), win_pitch(T.wh), win_s_hv(T.ww, T.wh)};
  const int ep = win_pitch(T.ww);
  const int hv = win_hv(ep, T.wh);
  const int hv2 = 2 * hv;                                                     // VD part of the window
  const int eb = -(T.wy0 * ep + T.wx0);                                       // event-window origin
  const int nbg = T.nbg;

  // ---------------- reverse of iteration k ----------------
  if (REV && !(KO(64))) {   // dq3 was zeroed before the stage arrived
    // lane descriptors, prefetched a bundle ahead (LDn: this warp's next bundle's)
    const uint32_t* LDn = P.ldesc + ((size_t)T.b0 + warp + NW) * 32 + lane;
    uint32_t ldn = ld_first;   // the first one was loaded before the stage wait
    for (int lb = warp; lb < T.nb; lb += NW) {
      const int4 bi = St.bi[lb];
      const uint32_t pw = St.pw[lb * 32 + lane];
      const uint32_t ld = ldn;
      if (lb + NW < nbg) ldn = __ldg(LDn);
      LDn += NW * 32;
      if (lb < nbg) {
        Lane L;
        lane_from_desc(bi, pw, ld, L);
        const int sl = lb * 32 + lane;
        const size_t gsl = (size_t)T.b0 * 32 + sl;
        float w = St.w[sl];
        const float2 mv = ld_stream2(&P.mv[gsl], pol);
        float m = mv.x, v = mv.y;
        const float p = ld_stream(&P.pp[gsl], pol);
        const float q = L.valid ? St.q[L.tree - t_lo] : 0.f;
        double c = 0.0;
        if (L.valid && !(KO(8))) {
          const short4 e = St.sxy[L.sub - s_lo];
          c = path_cost(St.S, W, X, Y, L.pw, e.x, e.y, e.z, e.w, A);
        }
        // softmax backward over the sub-net: with c_h the head's c and dd = c - c_h (fp64
        // difference, then fp32), sum_k p_k c_k = c_h + sa where sa = sum_k p_k dd_k (sum_k p_k = 1
        // up to ~1e-7), so dw_i = (p_i / t) q (dd_i - sa) and the head adds c_h + sa to dq_tree
        // (2^-32 fixed point): no cross-lane reduction over the tree's lanes.
        const double ch = __shfl_sync(kFull, c, L.head);
        const float dd = (float)(c - ch);
        float sa = seg_reduce(p * dd, L.lane, L.end, Sum());
        sa = __shfl_sync(kFull, sa, L.head);
        const float dw = L.valid ? p * A.inv_t * q * (dd - sa) : 0.f;
        if (L.valid && L.lane == L.head && (L.pw & kMultiTree))
          dq_add(dq3, L.tree - T.tree0, __double2ll_rn((c + (double)sa) * kDqScale));
        if (L.valid) {
          adam_update(w, m, v, dw, A);
          St.w[sl] = w;
          st_stream2(&P.mv[gsl], make_float2(m, v), pol);
        }
      } else if (__any_sync(kFull, pw & kMultiTree)) {
        // singleton bundle: c of a straight path (one segment, no turning point); p = 1.  Only dq
        // comes out of it, and only a multi-tree net's dq is used: bundles without one are skipped
        const bool valid = (pw & 7u) != kPad;
        const bool isv = (pw & 7u) == kStraightV;
        const int tree = bi.z + (int)((pw >> kTreeShift) & kTreeMask);
        double c = 0.0;
        if (valid && !(KO(8))) {
          const short4 e = St.sxy[bi.y + lane - s_lo];
          const int ia = isv ? W.v(e.x, e.y) : W.h(e.x, e.y);
          const int ib = isv ? W.v(e.x, e.w) : W.h(e.z, e.y);
          c = (St.S[ib] - St.S[ia]) + A.a_wl_d * (double)((e.z - e.x) + (e.w - e.y));
        }
        const uint32_t th = __ballot_sync(kFull, (pw & kTreeHead) || !valid) | 1u;
        const uint32_t le = kFull >> (31 - lane);
        const uint32_t trest = th & ~le;
        const int tend = trest ? (__ffs(trest) - 2) : 31;
        // each c rounded to the 2^-32 fixed point of dq BEFORE the tree-run sum: the run's split over
        // singleton bundles depends on the tile (and so on the rank count), integer sums do not
        const long long pc = seg_reduce(valid ? __double2ll_rn(c * kDqScale) : 0ll, lane, tend, Sum());
        if (valid && ((th >> lane) & 1u)) dq_add(dq3, tree - T.tree0, pc);
      }
    }
  }
  // the net level's tree Adam moments (one dependent global round trip on that phase's critical
  // path), loaded now: their latency hides behind the barrier and the dq reductions, and the
  // reverse's registers are dead here
  float mt_pre = 0.f, vt_pre = 0.f;
  (void)mt_pre; (void)vt_pre;
#if DGR_NL_EARLY
  if (REV && tid < T.nmn && mte != kNoTreeLane) {
    const int jg = T.tree0 + (int)(mte & 1023u);
    mt_pre = __ldcg(P.mt + jg);
    vt_pre = __ldcg(P.vt + jg);
  }
#endif
  if (REV && !(KO(64))) {
    __syncthreads();
  }
  stamp(P, (int)blockIdx.x - P.ntiles_slow - P.ngen_blocks, 2);

  // the forward's first lane descriptor, loaded before the net level (its latency hides there)
  const uint32_t ld_fwd = (FWD && warp < nbg) ? __ldg(P.ldesc + (size_t)T.b0 * 32 + warp * 32 + lane) : 0u;
  // ---------------- net level (one thread per net), event window cleared alongside ----------------
  if (FWD) {
    int4* z = reinterpret_cast<int4*>(ev_s);   // the S window is free after the reverse
    for (int i = tid; i < (3 * hv) / 4; i += NT) z[i] = make_int4(0, 0, 0, 0);
  }
  // the tile's nets with >= 2 trees, a lane per tree (a lone tree has q = 1 and du = 0 always: its
  // logit and Adam state never change, and its q = 1 arrives with the stage).  A net's trees are
  // consecutive lanes of one warp; its sums run over them in tree order (shuffles), the arithmetic of
  // the per-net loops of the slow path, so a net computes the same whichever tile it lands in.
  if (tid < ((KO(128)) ? 0 : T.nmn)) {   // whole warps (nmn is a multiple of 32)
    const uint32_t e = mte;
    const bool tv = e != kNoTreeLane;
    const int jr = (int)(e & 1023u);                    // tree, relative to the tile's first
    const int j = T.tree0 + jr - t_lo;                  // stage index
    const int nrel = (int)((e >> 10) & 2047u);           // net, relative to the tile's first
    const uint32_t hm = __ballot_sync(kFull, !tv || (e >> 31));
    const uint32_t le = kFull >> (31 - lane);
    const int head = 31 - __clz(hm & le);
    const uint32_t rest = hm & ~le;
    const int end = rest ? (__ffs(rest) - 2) : 31;
#if DGR_NL_EARLY
    // the tree's Gumbel noise first: independent of the reverse, it overlaps the Adam chain
    const uint32_t wd = (FWD && tv) ? twd[tid] : 0u;   // drawn at the tile's entry
    (void)nrel;
#endif
    if (REV) {
      // du_j = (q_j/t)(dq_j - sum_l q_l dq_l / sum_l q_l); Adam on w_tree (iteration k)
      const double ql = tv ? (double)St.q[j] : 0.0;
      const double qd = tv ? ql * dq_get(dq3, jr) : 0.0;
      double sq = 0.0, sw = 0.0;
      for (int k = 0; __any_sync(kFull, head + k <= end); ++k) {
        const int src = min(head + k, 31);
        const double a = __shfl_sync(kFull, qd, src), b = __shfl_sync(kFull, ql, src);
        if (head + k <= end) { sq += a; sw += b; }
      }
      sq /= sw;
      if (tv) {
        const double du = (double)St.q[j] * (double)A.inv_t * (dq_get(dq3, jr) - sq);
        const int jg = j + t_lo;
#if DGR_NL_EARLY
        float w = St.wt[j], m = mt_pre, v = vt_pre;
#else
        float w = St.wt[j], m = P.mt[jg], v = P.vt[jg];
#endif
        adam_update(w, m, v, (float)du, A);
        St.wt[j] = w;
        P.wt[jg] = w; P.mt[jg] = m; P.vt[jg] = v;
      }
    }
    if (FWD) {
      // q_j = softmax over the net's trees of (w_j + g_j)/t, iteration k_next (noise stream 1, keyed on
      // the global tree id: plan order = CSR order, else from net_gtree)
      float z = -INFINITY;
#if DGR_NL_EARLY
      if (tv) z = (St.wt[j] + gumbel_word(wd)) * A.inv_t;
#else
      const int jh = __shfl_sync(kFull, j, head);
      if (tv) {
        const int64_t gj = P.tree_base + (P.perm_id ? (int64_t)(t_lo + j) : (int64_t)__ldg(&P.net_gtree[T.net0 + nrel]) + (j - jh));
        const uint4 r = philox_rk(make_uint4((uint32_t)(gj >> 2), (uint32_t)(gj >> 34), (uint32_t)A.k_next, 1u), P.rk);
        const uint32_t wd = (gj & 3) == 0 ? r.x : (gj & 3) == 1 ? r.y : (gj & 3) == 2 ? r.z : r.w;
        z = (St.wt[j] + gumbel_word(wd)) * A.inv_t;
      }
#endif
      float zmax = -INFINITY;
      for (int k = 0; __any_sync(kFull, head + k <= end); ++k) {
        const float a = __shfl_sync(kFull, z, min(head + k, 31));
        if (head + k <= end) zmax = fmaxf(zmax, a);
      }
      const float ez = tv ? FEXP(z - zmax) : 0.f;
      float sum = 0.f;
      for (int k = 0; __any_sync(kFull, head + k <= end); ++k) {
        const float a = __shfl_sync(kFull, ez, min(head + k, 31));
        if (head + k <= end) sum += a;
      }
      if (tv) {
        const float q = ez / sum;
        St.q[j] = q;
        P.q[j + t_lo] = q;
      }
    }
  }
  if (FWD && nbg > 0 && !(KO(2))) tile_noise<NT, true>(P, T, (uint32_t)A.k_next, gp);   // path noise (stream 0)
  __syncthreads();
  stamp(P, (int)blockIdx.x - P.ntiles_slow - P.ngen_blocks, 3);

  // ---------------- forward of iteration k_next ----------------
  if (FWD) {
    const uint32_t ev_base = smem_u32(ev_s);
    const int gsh = noise_shift(P, T);
    // lane descriptors, prefetched a bundle ahead (LDn: this warp's next bundle's)
    const uint32_t* LDn = P.ldesc + ((size_t)T.b0 + warp + NW) * 32 + lane;
    uint32_t ldn = ld_fwd;
    for (int lb = warp; lb < T.nb; lb += NW) {
      const int4 bi = St.bi[lb];
      const uint32_t pw = St.pw[lb * 32 + lane];
      const uint32_t ld = ldn;
      if (lb + NW < nbg) ldn = __ldg(LDn);
      LDn += NW * 32;
      if (lb < nbg) {
        Lane L;
        lane_from_desc(bi, pw, ld, L);
        const int sl = lb * 32 + lane;
        const float w = St.w[sl];
        const float g = L.valid ? gumbel_word(__float_as_uint(gp[(ld & 0x7FFu) + gsh])) : 0.f;   // the lane's word, by its tile noise offset
        const float p = softmax_from_noise(L, w, g, A.inv_t);
        st_stream(&P.pp[(size_t)T.b0 * 32 + sl], p, pol);
        const float q = L.valid ? St.q[L.tree - t_lo] : 0.f;
        const int vq = L.valid ? __float2int_rn(q * p * kFixScale) : 0;
        if (L.valid && !(KO(4))) {
          // the candidate's own demand events in the Z(o, m) form (see path_cost): seg 1 from p0
          // to m on line q0, seg 2 from q0 to q1 on line m, seg 3 from m to p1 on line q1, each
          // +v at its lower and -v at its upper end, plus its turning points.  No cross-lane collapse: lanes of one
          // sub-net that share a corner cell meet in the shared-memory reduction.
          const short4 e = St.sxy[L.sub - s_lo];
          const int o = L.pw & 1, ntp = (L.pw >> 1) & 3, m = (int)(L.pw >> 16);
          // the event window's fields are row-major: cell (x, y) at (y - wy0) ww + x - wx0.  In the
          // Z(o, m) form a cell (a, b) of orientation o (a along the primary lines) is at a A + b B
          // with (A, B) = (1, ww) for o = 0 and (ww, 1) for o = 1, so the segment ends of one line
          // are ordered like their cell indices
          // (the sub-net's end cells need no orientation; a step along the primary lines is A_)
          const int A_ = o ? ep : 1;
          const int p0 = o ? e.y : e.x, p1 = o ? e.w : e.z;
          const int cp0 = e.y * ep + e.x + eb, cp1 = e.w * ep + e.z + eb;
          const int cm0 = cp0 + (m - p0) * A_, cm1 = cp1 + (m - p1) * A_;
          const int fP = o ? hv : 0, fS = hv - fP;   // fields of the primary / secondary lines
          // each segment: +v at its lower end, -v at its upper end (nothing if zero-length)
          const int v1 = cm0 != cp0 ? vq : 0, v2 = cm1 != cm0 ? vq : 0, v3 = cp1 != cm1 ? vq : 0;
#if !defined(DGR_EXP_SKIP_EVENTS)   // (timing experiments only: results invalid when defined)
#if !defined(DGR_EXP_SKIP_CORNERS)
          red_shared_add(ev_base + 4u * (fP + min(cp0, cm0)), v1);
#endif
          red_shared_add(ev_base + 4u * (fP + max(cp0, cm0)), -v1);
          red_shared_add(ev_base + 4u * (fS + min(cm0, cm1)), v2);
          red_shared_add(ev_base + 4u * (fS + max(cm0, cm1)), -v2);
          red_shared_add(ev_base + 4u * (fP + min(cm1, cp1)), v3);
#if !defined(DGR_EXP_SKIP_CORNERS)
          red_shared_add(ev_base + 4u * (fP + max(cm1, cp1)), -v3);
#endif
          red_shared_add(ev_base + 4u * (hv2 + cm0), ntp >= 1 ? vq : 0);   // turning points
          red_shared_add(ev_base + 4u * (hv2 + cm1), ntp == 2 ? vq : 0);
#else
          if (vq == 123456789) red_shared_add(ev_base + 4u * (fP + cp0 + cm0 + cm1 + cp1 + fS + v1 + v2 + v3), 1);
#endif
        }
      } else {
        // singleton bundle: pi = q; +pi where the segment starts, -pi where it ends
        const bool valid = (pw & 7u) != kPad;
        if (valid && !(KO(4))) {
          const bool isv = (pw & 7u) == kStraightV;
          const int tree = bi.z + (int)((pw >> kTreeShift) & kTreeMask);
          const float q = St.q[tree - t_lo];
          const int vq = __float2int_rn(q * kFixScale);
          const short4 e = St.sxy[bi.y + lane - s_lo];
          const int ia = e.y * ep + e.x + eb + (isv ? hv : 0);   // row-major event fields
          const int ib = (isv ? e.w * ep + e.x + hv : e.y * ep + e.z) + eb;
          red_shared_add(ev_base + 4u * ia, vq);
          red_shared_add(ev_base + 4u * ib, -vq);
        }
      }
    }
  }
  __syncthreads();
  stamp(P, (int)blockIdx.x - P.ntiles_slow - P.ngen_blocks, 4);
  // write back the tile's group slot state with bulk stores (asynchronous; readers wait on the group)
  if (tid == 0 && nbg > 0) {
    fence_proxy_async();
    const size_t s0 = (size_t)T.b0 * 32;
    const uint32_t gslot_bytes = (uint32_t)nbg * 128u;
    if (REV) bulk_s2g_stream(P.wp + s0, St.w, gslot_bytes, policy_stream());
    bulk_commit();
  }
  if (FWD && !(KO(1))) {
    // flush the window once, then the tile's shares of E[TP] and of the border deficit summed in
    // warp order into the exchange buffer's counters
    long long etp = 0, bdef = 0;
    flush_window<NT>(P, A, T.wx0, T.wy0, T.ww, T.wh, ep, hv, ev_s, etp, bdef);
    etp = warp_sum_ll(etp);
    bdef = warp_sum_ll(bdef);
    long long* part = reinterpret_cast<long long*>(dq3);   // free after the net level
    if (lane == 0) { part[2 * warp] = etp; part[2 * warp + 1] = bdef; }
    __syncthreads();
    if (tid == 0) {
      long long a = 0, b = 0;
#pragma unroll
      for (int w = 0; w < NW; ++w) { a += part[2 * w]; b += part[2 * w + 1]; }
      if (a | b) {
        atomicAdd(reinterpret_cast<unsigned long long*>(P.acc), (unsigned long long)a);
        atomicAdd(reinterpret_cast<unsigned long long*>(P.acc + 1), (unsigned long long)b);
      }
    }
  }
}

// ------------------------------------------------------------------------------------------
// General nets (row f4', reading Q14c): any rectilinear candidates (monotone staircases ...), groups
// of up to kGenMaxGroup, any candidate order.  One warp per net, from explicit segment and
// turning-point lists, against S and the difference arrays in global memory; a group is processed
// in chunks of 32 lanes.  Same formulas as the tile path: c_i (Eqs. (9)-(12) chain rule, reading
// Q3), softmax backward with differences to the group's first candidate, Adam, tree level, noise
// keyed on the global noise / tree index (Q7), +-pi segment events and folded turning points.
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ double gen_cost(const KParams& P, const StepArgs& A, int gp) {
  const int X = P.X, Y = P.Y;
  double c = 0.0, tp = 0.0;
  int wl = 0;
  // (unrolled: the segment records and then their S values load in parallel, not one dependent
  // pair of L2 round trips per segment)
#pragma unroll 4
  for (int q = P.gp_seg_off[gp]; q < P.gp_seg_off[gp + 1]; ++q) {
    const short4 g = P.gseg[q];   // {dir, line, lo, hi}: edges [lo, hi) of the line
    const double* S = g.x == 0 ? P.SH + (size_t)g.y * P.XP : P.SVT + (size_t)g.y * P.YP;
    c += S[g.w] - S[g.z];
    wl += g.w - g.z;
  }
  const int t0 = P.gp_tp_off[gp], t1 = P.gp_tp_off[gp + 1];
#pragma unroll 4
  for (int q = t0; q < t1; ++q) {   // the (clipped) edges left / right and below / above the cell
    const short2 v = P.gtp[q];
    const double* SH = P.SH + (size_t)v.y * P.XP;
    const double* SV = P.SVT + (size_t)v.x * P.YP;
    tp += (SH[v.x + (v.x < X - 1)] - SH[v.x - (v.x > 0)]) + (SV[v.y + (v.y < Y - 1)] - SV[v.y - (v.y > 0)]);
  }
  return c + A.beta_d * tp + A.a_wl_d * (double)wl + A.via_d * (double)(t1 - t0);
}

// demand events of general path gp with weight v (2^-24): +-v at each segment's ends, folded turning points
__device__ __forceinline__ void gen_events(const KParams& P, const StepArgs& A, int gp, int v, long long& etp, long long& bdef) {
  if (v == 0) return;
  const long long vs = (long long)v << kGridShift;
#pragma unroll 4
  for (int q = P.gp_seg_off[gp]; q < P.gp_seg_off[gp + 1]; ++q) {
    const short4 g = P.gseg[q];
    long long* diff = g.x == 0 ? P.dH + (size_t)g.y * P.X : P.dVT + (size_t)g.y * P.Y;
    red64(diff + g.z, vs);
    red64(diff + g.w, -vs);
  }
#pragma unroll 4
  for (int q = P.gp_tp_off[gp]; q < P.gp_tp_off[gp + 1]; ++q) {
    const short2 t = P.gtp[q];
    tp_fold_global(P, A, t.x, t.y, v, etp, bdef);
  }
}

__device__ __forceinline__ float warp_sum_f(float v) {
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(kFull, v, off);
  return v;
}
__device__ __forceinline__ float warp_max_f(float v) {
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) v = fmaxf(v, __shfl_xor_sync(kFull, v, off));
  return v;
}

template <bool REV, bool FWD>
__device__ __forceinline__ void gen_net(const KParams& P, const StepArgs& A, int gn, long long& etp, long long& bdef) {
  const int lane = threadIdx.x & 31;
  const int2 nd = P.gnet[gn];   // {first gtree, trees}
  if (REV) {   // reverse of iteration k
    for (int g = nd.x; g < nd.x + nd.y; ++g) {
      const int4 gt = P.gtree[g];   // {local tree, first gsub, sub-nets, multi-tree}
      const float q = P.q[gt.x];
      // dq_j = sum over the tree's sub-nets of sum_k p_k c_k (2^-32 fixed point: exact, any order).
      // Lone straight paths (p = 1: their c goes to dq as is) a lane each, then the groups
      long long dq = 0;
      for (int s = gt.y + lane; s < gt.y + gt.z; s += 32) {
        const GSub G = P.gsub[s];
        if (G.nid < 0) dq += __double2ll_rn(gen_cost(P, A, G.gp) * kDqScale);
      }
      dq = warp_sum_ll(dq);         // (lane 0 holds the total)
      for (int s = gt.y; s < gt.y + gt.z; ++s) {
        const GSub G = P.gsub[s];
        if (G.nid < 0) continue;
        double c0 = 0.0, cl = 0.0;  // the group's first c; this lane's c of the first chunk
        float sa = 0.f;             // sum_k p_k (c_k - c_0)
        for (int b = 0; b < G.n; b += 32) {
          const int i = b + lane;
          const bool v = i < G.n;
          const double c = v ? gen_cost(P, A, G.gp + i) : 0.0;
          if (b == 0) { c0 = __shfl_sync(kFull, c, 0); cl = c; }
          sa += v ? P.pp[G.slot + i] * (float)(c - c0) : 0.f;
        }
        sa = warp_sum_f(sa);
        for (int b = 0; b < G.n; b += 32) {
          const int i = b + lane;
          if (i < G.n) {
            const double c = b == 0 ? cl : gen_cost(P, A, G.gp + i);
            const int sl = G.slot + i;
            const float p = P.pp[sl];
            const float dw = p * A.inv_t * q * ((float)(c - c0) - sa);   // (p_i/t) q (dd_i - sum_k p_k dd_k)
            float w = P.wp[sl];
            float2 mv = P.mv[sl];
            adam_update(w, mv.x, mv.y, dw, A);
            P.wp[sl] = w;
            P.mv[sl] = mv;
          }
        }
        if (lane == 0) dq += __double2ll_rn((c0 + (double)sa) * kDqScale);
      }
      if (lane == 0) P.gdq[g] = dq;
    }
    __syncwarp();
  }
  if (lane == 0) {   // tree level: du_j, Adam on w_tree (k); q_j of k+1 (noise stream 1)
    const int g0 = nd.x, g1 = nd.x + nd.y;
    if (REV && nd.y > 1) {
      double sq = 0.0, sw = 0.0;
      for (int g = g0; g < g1; ++g) {
        const double ql = (double)P.q[P.gtree[g].x];
        sq += ql * ((double)P.gdq[g] * kDqInv);
        sw += ql;
      }
      sq /= sw;
      for (int g = g0; g < g1; ++g) {
        const int j = P.gtree[g].x;
        const double du = (double)P.q[j] * (double)A.inv_t * ((double)P.gdq[g] * kDqInv - sq);
        float w = P.wt[j], m = P.mt[j], v = P.vt[j];
        adam_update(w, m, v, (float)du, A);
        P.wt[j] = w; P.mt[j] = m; P.vt[j] = v;
      }
    }
    if (FWD && nd.y > 1) {   // a lone tree keeps q = 1
      float zmax = -INFINITY;
      for (int g = g0; g < g1; ++g) {
        const int j = P.gtree[g].x;
        zmax = fmaxf(zmax, (P.wt[j] + gumbel(P.seed, (uint64_t)(P.tree_base + P.gtree[g].w), (uint32_t)A.k_next, 1u)) * A.inv_t);
      }
      float sum = 0.f;
      for (int g = g0; g < g1; ++g) {
        const int j = P.gtree[g].x;
        sum += FEXP((P.wt[j] + gumbel(P.seed, (uint64_t)(P.tree_base + P.gtree[g].w), (uint32_t)A.k_next, 1u)) * A.inv_t - zmax);
      }
      for (int g = g0; g < g1; ++g) {
        const int j = P.gtree[g].x;
        P.q[j] = FEXP((P.wt[j] + gumbel(P.seed, (uint64_t)(P.tree_base + P.gtree[g].w), (uint32_t)A.k_next, 1u)) * A.inv_t - zmax) / sum;
      }
    }
  }
  __syncwarp();
  if (FWD) {   // forward of iteration k+1
    for (int g = nd.x; g < nd.x + nd.y; ++g) {
      const int4 gt = P.gtree[g];
      const float q = P.q[gt.x];
      for (int s = gt.y + lane; s < gt.y + gt.z; s += 32) {   // lone straight paths (pi = q), a lane each
        const GSub G = P.gsub[s];
        if (G.nid < 0) gen_events(P, A, G.gp, __float2int_rn(q * kFixScale), etp, bdef);
      }
      for (int s = gt.y; s < gt.y + gt.z; ++s) {
        const GSub G = P.gsub[s];
        if (G.nid < 0) continue;
        // p_i = softmax over the group of (w_i + g_i) / t: the maximum, then the sum, then p
        float zl = -INFINITY, zmax = -INFINITY;
        for (int b = 0; b < G.n; b += 32) {
          const int i = b + lane;
          const float z = i < G.n ? (P.wp[G.slot + i] + gumbel(P.seed, (uint64_t)(P.nid_base + G.nid + i), (uint32_t)A.k_next, 0u)) * A.inv_t
                                  : -INFINITY;
          if (b == 0) zl = z;
          zmax = fmaxf(zmax, z);
        }
        zmax = warp_max_f(zmax);
        float sum = 0.f;
        for (int b = 0; b < G.n; b += 32) {
          const int i = b + lane;
          const float z = b == 0 ? zl : (i < G.n ? (P.wp[G.slot + i] + gumbel(P.seed, (uint64_t)(P.nid_base + G.nid + i), (uint32_t)A.k_next, 0u)) * A.inv_t : -INFINITY);
          sum += i < G.n ? FEXP(z - zmax) : 0.f;
        }
        sum = warp_sum_f(sum);
        for (int b = 0; b < G.n; b += 32) {
          const int i = b + lane;
          if (i < G.n) {
            const float z = b == 0 ? zl : (P.wp[G.slot + i] + gumbel(P.seed, (uint64_t)(P.nid_base + G.nid + i), (uint32_t)A.k_next, 0u)) * A.inv_t;
            const float p = FDIV(FEXP(z - zmax), sum);
            P.pp[G.slot + i] = p;
            gen_events(P, A, G.gp + i, __float2int_rn(q * p * kFixScale), etp, bdef);
          }
        }
      }
    }
  }
}

template <bool REV, bool FWD>
__device__ __forceinline__ void gen_block(const KParams& P, const StepArgs& A, int gb) {
  const int warp = threadIdx.x >> 5;
  long long etp = 0, bdef = 0;
  for (int gn = gb * kGenWarps + warp; gn < P.ngen; gn += P.ngen_blocks * kGenWarps) gen_net<REV, FWD>(P, A, gn, etp, bdef);
  if (FWD) {
    etp = warp_sum_ll(etp);
    bdef = warp_sum_ll(bdef);
    if ((threadIdx.x & 31) == 0 && (etp | bdef)) {   // exact integers: any order gives the same sums
      atomicAdd(reinterpret_cast<unsigned long long*>(P.acc), (unsigned long long)etp);
      atomicAdd(reinterpret_cast<unsigned long long*>(P.acc + 1), (unsigned long long)bdef);
    }
  }
}

// (a) one tile per CTA: the whole tile arrives by bulk copies on one mbarrier; the event window
// and noise alias the S window.  4 CTAs per SM overlap one CTA's copies with the others' math.
#ifndef DGR_BTHREADS
#define DGR_BTHREADS 256
#endif
constexpr int kBThreads = DGR_BTHREADS;
#ifndef DGR_LSU_STAGE
#define DGR_LSU_STAGE 2   // stage: 1-D arrays by bulk copies + S window by cp.async (2), all by
                          // cp.async (1), all by cp.async.bulk on an mbarrier (0)
#endif
#ifndef DGR_BPERSM
#define DGR_BPERSM 5
#endif
constexpr int kBPerSM = DGR_BPERSM;
constexpr size_t kTailBytes = 12 * kPipeTrees + 16 + 4 * kBThreads;   // dq limbs, mbarrier, tree noise words
constexpr size_t kBSmemBytes = (StageLayout::bytes + kTailBytes) > kSmemBytes ? (StageLayout::bytes + kTailBytes) : kSmemBytes;
static_assert(kGpOffset + 4 * 32 * kTargetBundles + 32 <= 2 * 8 * (kWinMax + kWinPad), "event window + path noise must fit the S window");

template <bool REV, bool FWD>
__global__ void __launch_bounds__(kBThreads, kBPerSM) tile_bulk(KParams P, StepArgs A) {
  extern __shared__ __align__(128) unsigned char smem[];
  Stage St(smem);
  int* dq3 = reinterpret_cast<int*>(smem + StageLayout::bytes);
  uint64_t* bar = reinterpret_cast<uint64_t*>(dq3 + 3 * kPipeTrees);
  griddep_launch();
  if ((int)blockIdx.x < P.ntiles_slow) {   // global tiles first: the longest CTAs start earliest
    griddep_wait();
    if (!(KO(512))) slow_tile<REV, FWD>(P, A, P.tiles_slow[blockIdx.x], smem);   // (knock-out 512: timing only)
    return;
  }
  if ((int)blockIdx.x < P.ntiles_slow + P.ngen_blocks) {   // general nets (row f4'): a warp per net
    griddep_wait();
    gen_block<REV, FWD>(P, A, (int)blockIdx.x - P.ntiles_slow);
    return;
  }
  int* ev_s = reinterpret_cast<int*>(St.S);
  float* gp = reinterpret_cast<float*>(reinterpret_cast<unsigned char*>(St.S) + kGpOffset);
  const int tix = (int)blockIdx.x - P.ntiles_slow - P.ngen_blocks;
  const TileDesc T = P.tiles[tix];
  stamp(P, tix, 0);
  if ((KO(256)) && threadIdx.x == 0 && tix < kProfTiles) {
    unsigned sm, gt_lo;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
    long long gt;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt));
    g_tile_prof[tix * 8 + 6] = sm;
    g_tile_prof[tix * 8 + 7] = gt;
    (void)gt_lo;
  }
  if (threadIdx.x == 0) {
    mbar_init(bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  for (int i = threadIdx.x; i < 3 * kPipeTrees; i += kBThreads) dq3[i] = 0;
  // the reverse's first lane descriptor (plan data: no dependence on the previous kernels), loaded
  // now so that its latency hides behind the stage
  const int wid = threadIdx.x >> 5;
  const uint32_t ld_first = (REV && wid < T.nbg) ? __ldg(P.ldesc + (size_t)T.b0 * 32 + wid * 32 + (threadIdx.x & 31)) : 0u;
  // this thread's tree lane of the net level (plan data), likewise
  const uint32_t mte = (int)threadIdx.x < T.nmn ? __ldg(P.mnets + T.mn0 + threadIdx.x) : kNoTreeLane;
  __syncthreads();
  griddep_wait();   // S, logits, q and the event grids come from the previous kernels
  uint32_t* twd = reinterpret_cast<uint32_t*>(bar + 2);   // the net level's tree noise words
#if DGR_LSU_STAGE == 2
  // the eight 1-D arrays by bulk copies (8 per tile: few and large), the S window by cp.async
  if (threadIdx.x < 32) {
    issue_tile_loads<REV>(P, T, smem, bar, false);
    // the trees' Adam moments are read by the net level (one dependent chain per net, the
    // phase's critical path): bring them to L2 with the stage (DGR_PF bit 1; bit 0 also the slots')
    if (REV && (P.pf & 3)) prefetch_tile(P, T, (P.pf & 1) != 0);
  }
  lsu_tile_loads<REV, kBThreads>(P, T, smem, false);
  // the net level's tree noise (stream 1, keyed on the global tree id: plan data and the iteration
  // only), drawn while the stage is in flight: off that phase's critical path.  Raw
  // Philox words, one per tree lane, read back by the same thread.
  if (FWD && (int)threadIdx.x < T.nmn) {   // whole warps (nmn is a multiple of 32)
    const int lane = threadIdx.x & 31;
    const bool tv = mte != kNoTreeLane;
    const int j = T.tree0 + (int)(mte & 1023u) - (T.tree0 & ~3);   // stage index, as in the net level
    const uint32_t hm = __ballot_sync(kFull, !tv || (mte >> 31));
    const int head = 31 - __clz(hm & (kFull >> (31 - lane)));
    const int jh = __shfl_sync(kFull, j, head);
    if (tv) {
      const int nrel = (int)((mte >> 10) & 2047u);
      const int64_t gj = P.tree_base + (P.perm_id ? (int64_t)(T.tree0 + (int)(mte & 1023u))
                                                  : (int64_t)__ldg(&P.net_gtree[T.net0 + nrel]) + (j - jh));
      const uint4 r = philox_rk(make_uint4((uint32_t)(gj >> 2), (uint32_t)(gj >> 34), (uint32_t)A.k_next, 1u), P.rk);
      twd[threadIdx.x] = (gj & 3) == 0 ? r.x : (gj & 3) == 1 ? r.y : (gj & 3) == 2 ? r.z : r.w;
    }
  }
  asm volatile("cp.async.wait_group 0;" ::: "memory");
  mbar_wait(bar, 0u);
  __syncthreads();
#elif DGR_LSU_STAGE
  if (threadIdx.x < 32 && (P.pf & 1)) prefetch_tile(P, T);
  lsu_tile_loads<REV, kBThreads>(P, T, smem);
  asm volatile("cp.async.wait_group 0;" ::: "memory");
  __syncthreads();
#else
  if (threadIdx.x < 32) {
    issue_tile_loads<REV>(P, T, smem, bar);
    if (P.pf & 1) prefetch_tile(P, T);
  }
  mbar_wait(bar, 0u);
#endif
  stamp(P, tix, 1);
  if (!(KO(16))) process_tile<REV, FWD, kBThreads>(P, A, T, St, ev_s, gp, dq3, ld_first, mte, twd);
  if (KO(256)) __syncthreads();   // (diagnostics: the flush of every warp is done)
  stamp(P, tix, 5);
  if (threadIdx.x == 0) bulk_wait_read();   // the stage must outlive the bulk stores' reads
}

// ------------------------------------------------------------------------------------------
// KG: one CTA per line (Y H-rows, then X V-columns).  Scan of the difference array gives the
// wire demand W; d = (W + beta (VD_a + VD_b)) 2^-24 (Eq. (10), reading Q3); overflow cost
// f(d - cap) (Eq. (9), reading Q2); G = dcost/dd = a3 f'(d - cap); S = exclusive prefix of G (fp64).
// The line's difference and turning-point entries are cleared for the next forward.
// ------------------------------------------------------------------------------------------
constexpr int kGThreads = 32 * kKgWarps;
#ifndef DGR_KG_ITEMS
#define DGR_KG_ITEMS 4
#endif
constexpr int kGItems = DGR_KG_ITEMS;

template <typename T>
__device__ __forceinline__ T block_exclusive_scan(T v, T* sh, T* total) {
  // sh: >= 32 entries
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  T x = v;
#pragma unroll
  for (int off = 1; off < 32; off <<= 1) {
    const T o = __shfl_up_sync(kFull, x, off);
    if (lane >= off) x += o;
  }
  if (lane == 31) sh[wid] = x;
  __syncthreads();
  if (wid == 0) {
    T y = lane < nw ? sh[lane] : T(0);
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
      const T o = __shfl_up_sync(kFull, y, off);
      if (lane >= off) y += o;
    }
    if (lane < nw) sh[lane] = y;   // inclusive warp totals
  }
  __syncthreads();
  const T before = wid ? sh[wid - 1] : T(0);
  *total = sh[nw - 1];
  __syncthreads();
  return before + x - v;
}

// warp-inclusive scan (shuffles)
template <typename T>
__device__ __forceinline__ T warp_inclusive_scan(T x, int lane) {
#pragma unroll
  for (int off = 1; off < 32; off <<= 1) {
    const T o = __shfl_up_sync(kFull, x, off);
    if (lane >= off) x += o;
  }
  return x;
}

// Exclusive scan of a chunk of kGThreads * kGItems elements held "striped": thread t holds
// elements j * kGThreads + t (j < kGItems), so every global access is coalesced.  Warp scans of
// each item, then one warp scans the kGItems * NW warp totals (in position order), two barriers.
// The caller puts a barrier between two uses of the same sh.
template <typename T>
__device__ __forceinline__ void striped_exclusive_scan(T (&v)[kGItems], T* sh /* kGItems*32 */, T* total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  constexpr int NW = kGThreads / 32;
  static_assert(kGItems * NW <= 32, "one warp scans the segment totals");
  T inc[kGItems];
#pragma unroll
  for (int j = 0; j < kGItems; ++j) inc[j] = warp_inclusive_scan(v[j], lane);
  if (lane == 31) {
#pragma unroll
    for (int j = 0; j < kGItems; ++j) sh[j * NW + wid] = inc[j];
  }
  __syncthreads();
  if (wid == 0) {
    const T t = lane < kGItems * NW ? sh[lane] : T(0);
    const T x = warp_inclusive_scan(t, lane);
    if (lane < kGItems * NW) sh[lane] = x - t;        // exclusive prefix of the segment totals
    if (lane == kGItems * NW - 1) sh[32] = x;         // chunk total
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < kGItems; ++j) v[j] = sh[j * NW + wid] + inc[j] - v[j];   // exclusive
  *total = sh[32];
  // no trailing barrier: the caller separates reuses of sh (the next chunk of a line) by one
}

// The loss of the last KG launch (Eqs. (9), (11), (12)): sums of the per-line partials in line
// order (deterministic).  One CTA, launched once per dgr_step call after its last KG.
__global__ void __launch_bounds__(1024) kg_loss_kernel(KParams P, StepArgs A) {
  // fixed-shape tree reduction (strided thread sums, warp shuffles, warp totals in warp order):
  // deterministic, one pass, no block scans
  __shared__ double shs[32], shd[32];
  const int nl = P.X + P.Y, lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  griddep_wait();   // launched with PDL behind the last KG: its partials
  double s = 0.0, sd = 0.0;
  for (int i = threadIdx.x; i < nl; i += blockDim.x) {
    s += P.partial[i];
    sd += (double)P.lpart[i] * kGridInv;   // each line's sum of the demand (exact in 2^-40, ~1e4 tracks)
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    s += __shfl_down_sync(kFull, s, off);
    sd += __shfl_down_sync(kFull, sd, off);
  }
  if (lane == 0) { shs[wid] = s; shd[wid] = sd; }
  __syncthreads();
  if (wid == 0) {
    const int nw = blockDim.x >> 5;
    s = lane < nw ? shs[lane] : 0.0;
    sd = lane < nw ? shd[lane] : 0.0;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      s += __shfl_down_sync(kFull, s, off);
      sd += __shfl_down_sync(kFull, sd, off);
    }
    if (lane == 0) {
      // E[TP] = sum of the turning points (exact fixed point, the exchange buffer's counter); the
      // folded demand sums to E[WL] + beta sum_v VD_v deg(v) = E[WL] + beta (4 E[TP] - B)
      const double etp = (double)P.lsum[0] * kFixInv;
      const double bdef = (double)P.lsum[1] * kFixInv;
      const double ewl = sd - (double)A.beta * (4.0 * etp - bdef);
      const double via = (double)A.sqrt_l * etp;
      P.loss[0] = (double)A.a_wl * ewl + (double)A.a_via * via + (double)A.a_of * s;
      P.loss[1] = ewl;
      P.loss[2] = via;
      P.loss[3] = s;
      if (P.loss_host) {   // straight into the caller's pinned buffer (visible after the stream syncs)
        P.loss_host[0] = P.loss[0]; P.loss_host[1] = ewl; P.loss_host[2] = via; P.loss_host[3] = s;
      }
    }
  }
}

// f(x) and df/dx = df/dd of the overflow x = d - cap (Eq. (9), reading Q2) in fp32 (x itself in
// fp64: d comes from exact fixed point); relative error ~1e-6, well inside the 1e-4 bar, at a
// fraction of fp64 exp's cost
__device__ __forceinline__ void overflow_f(const StepArgs& A, double x, double& fv, double& fg) {
  const float xf = (float)x, sf = A.f_slope;
  switch (A.f_kind) {
    case 0: {   // sigmoid sigma(s x); stable for both signs
      const float e = FEXP(-fabsf(sf * xf));
      const float inv = FDIV(1.f, 1.f + e);
      fv = (sf * xf > 0.f) ? inv : e * inv;
      fg = sf * e * inv * inv;
      break;
    }
    case 1: fv = x > 0.0 ? x : 0.0; fg = x > 0.0 ? 1.0 : 0.0; break;        // ReLU
    case 2: fv = x > 0.0 ? x : (double)sf * x; fg = x > 0.0 ? 1.0 : (double)sf; break;   // LeakyReLU (Fig. 6)
    case 3: fv = exp((double)sf * x); fg = (double)sf * fv; break;          // exp (Fig. 6): fp64 range
    default: {                                                              // CELU (Fig. 6)
      const float e = expf(fminf(xf, 0.f) / sf);
      fv = x > 0.0 ? x : (double)(sf * (e - 1.f));
      fg = x > 0.0 ? 1.0 : (double)e;
    }
  }
}

#ifndef DGR_KG_MINB
#define DGR_KG_MINB 4
#endif
// One CTA per line (the launch has X + Y CTAs; CTA b would take lines b, b + gridDim.x, ... of a
// smaller grid), chunk by chunk: the next chunk's difference and capacity values are loaded into
// registers before the current one is scanned, so a long line's loads overlap its scans and
// barriers.  (A persistent grid of resident CTAs was measured 1% slower per iteration: it holds
// every SM slot until its last line, so the next KBF's CTAs cannot fill in behind it under PDL.)
__global__ void __launch_bounds__(kGThreads, DGR_KG_MINB) kg_kernel(KParams P, StepArgs A) {
  __shared__ long long shl[33];
  __shared__ double shd[33];
  __shared__ double shw[kKgWarps];
  __shared__ long long shwl[kKgWarps];
  griddep_launch();
  griddep_wait();   // the difference arrays are complete (the previous KBF / allreduce)
  // the rank's lines (SURVEY §8(e) refinement 2): H rows [kg_h0, kg_h1), then V columns [kg_v0, kg_v1)
  // (all of them on one GPU); slot b is line slot_line(b) (line ids: rows 0..Y-1, columns Y..Y+X-1)
  const int nhs = P.kg_h1 - P.kg_h0, nl = nhs + (P.kg_v1 - P.kg_v0), lane = threadIdx.x & 31;
  auto slot_line = [&](int b) { return b < nhs ? P.kg_h0 + b : P.Y + P.kg_v0 + (b - nhs); };
  if (blockIdx.x == 0 && threadIdx.x == 0) {   // E[TP], B of this forward, for the loss; cleared for the next
    P.lsum[0] = P.acc[0]; P.lsum[1] = P.acc[1];
    P.acc[0] = 0; P.acc[1] = 0;
  }
  auto line_len = [&](int l) { return l < P.Y ? P.X : P.Y; };
  auto line_diff = [&](int l) { return l < P.Y ? P.dH + (size_t)l * P.X : P.dVT + (size_t)(l - P.Y) * P.Y; };
  auto line_cap = [&](int l) { return l < P.Y ? P.capH + (size_t)l * P.X : P.capVT + (size_t)(l - P.Y) * P.Y; };
  long long v[kGItems];
  float cp[kGItems];
  auto load = [&](int l, int c0, long long (&vv)[kGItems], float (&cc)[kGItems]) {
    const int n = line_len(l);
    const long long* diff = line_diff(l);
    const float* cap = line_cap(l);
#pragma unroll
    for (int j = 0; j < kGItems; ++j) {
      const int pos = c0 + j * kGThreads + threadIdx.x;
      vv[j] = pos < n ? diff[pos] : 0;
      cc[j] = pos < n ? cap[pos] : 0.f;
    }
  };
  int slot = blockIdx.x, c0 = 0;
  if (slot >= nl) return;
  int line = slot_line(slot);
  load(line, 0, v, cp);
  long long carryW = 0, sumD = 0;   // sumD: sum over the line's edges of the demand (2^-40)
  double carryS = 0.0, of = 0.0;
  while (true) {
    const bool isH = line < P.Y;
    const int n = isH ? P.X : P.Y;
    const int ln = isH ? line : line - P.Y;
    long long* diff = line_diff(line);
    double* S = isH ? P.SH + (size_t)ln * P.XP : P.SVT + (size_t)ln * P.YP;
    float* dout = (isH ? P.dOutH : P.dOutVT) + (size_t)ln * n;
    // the next chunk of this CTA (the rest of this line, else its next line), prefetched
    int nslot = slot, nc0 = c0 + kGThreads * kGItems;
    if (nc0 >= n) { nslot += gridDim.x; nc0 = 0; }
    const int nline = nslot < nl ? slot_line(nslot) : -1;
    long long nv[kGItems];
    float ncp[kGItems];
    if (nslot < nl) load(nline, nc0, nv, ncp);
    long long totW;
    long long ex[kGItems];
#pragma unroll
    for (int j = 0; j < kGItems; ++j) ex[j] = v[j];
    striped_exclusive_scan(ex, shl, &totW);   // all reads of this chunk are done after its barrier
#pragma unroll
    for (int j = 0; j < kGItems; ++j) {
      const int pos = c0 + j * kGThreads + threadIdx.x;
      if (pos < n) diff[pos] = 0;   // cleared for the next forward
    }
    double g[kGItems];
#pragma unroll
    for (int j = 0; j < kGItems; ++j) {
      const int pos = c0 + j * kGThreads + threadIdx.x;
      double G = 0.0;
      if (pos < n - 1) {
        // inclusive prefix = demand of edge pos: W_e + beta (VD_a + VD_b) (Eq. (10), reading Q3)
        const long long D = carryW + ex[j] + v[j];
        sumD += D;
        const double d = (double)D * kGridInv;
        double fv, fg;
        overflow_f(A, d - (double)cp[j], fv, fg);   // overflow x = d - cap = -(cap - d)
        of += fv;
        G = (double)A.a_of * fg;
        if (A.store_d) dout[pos] = (float)d;
      } else if (pos == n - 1 && A.store_d) {
        dout[pos] = 0.f;
      }
      g[j] = G;
    }
    double totS;
    striped_exclusive_scan(g, shd, &totS);
#pragma unroll
    for (int j = 0; j < kGItems; ++j) {
      const int pos = c0 + j * kGThreads + threadIdx.x;
      if (pos < n) S[pos] = carryS + g[j];
    }
    carryW += totW;
    carryS += totS;
    if (nline != line) {
      // per-line partials of the overflow cost and the demand sum: warp sums, then thread 0 sums
      // the warps in order (deterministic); kg_loss_kernel sums the lines
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        of += __shfl_down_sync(kFull, of, off);
        sumD += __shfl_down_sync(kFull, sumD, off);
      }
      if (lane == 0) { shw[threadIdx.x >> 5] = of; shwl[threadIdx.x >> 5] = sumD; }
      __syncthreads();
      if (threadIdx.x == 0) {
        double tot = 0.0;
        long long td = 0;
#pragma unroll
        for (int w = 0; w < kKgWarps; ++w) { tot += shw[w]; td += shwl[w]; }
        P.partial[line] = tot;
        P.lpart[line] = td;
      }
      carryW = 0; sumD = 0; carryS = 0.0; of = 0.0;
    }
    if (nslot >= nl) break;
    __syncthreads();   // the next chunk reuses shl / shd / shw
    slot = nslot; line = nline; c0 = nc0;
#pragma unroll
    for (int j = 0; j < kGItems; ++j) { v[j] = nv[j]; cp[j] = ncp[j]; }
  }
}


// ------------------------------------------------------------------------------------------
// Induction (§4.5): KI1 argmax tree per net; KI2 top-p nucleus + route per sub-net of the
// chosen tree, integer rasterisation of the route; KI3 overflow metrics of Eq. (2)'s demand.
// ------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) ki_tree_kernel(KParams P) {
  const int n = blockIdx.x * blockDim.x + threadIdx.x;
  if (n >= P.n_nets_l) return;
  const int a = P.net_tree_off[n], b = P.net_tree_off[n + 1];
  int best = a;
  for (int j = a + 1; j < b; ++j) if (P.wt[j] > P.wt[best]) best = j;   // q_hat monotone in w
  for (int j = a; j < b; ++j) P.chosen[j] = (j == best);
  P.tree_choice[n] = (int32_t)(P.tree_base + P.net_gtree[n] + (best - a));   // global (CSR) tree id
}

__global__ void __launch_bounds__(256) ki_path_kernel(KParams P, float inv_t, float top_p) {
  const int b = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (b >= P.nb) return;
  Lane L;
  lane_setup(P, b, L);
  const size_t slot = (size_t)b * 32 + L.lane;
  const bool on = L.valid && P.chosen[L.tree];
  const float w = L.valid ? P.wp[slot] : -INFINITY;
  // rank by (w desc, index asc): p_hat = softmax(w/t) is monotone in w
  int rank = 0;
  for (int j = 0; j < 32; ++j) {
    const float wj = __shfl_sync(kFull, w, j);
    if (((L.gmask >> j) & 1u) && (wj > w || (wj == w && j < L.lane))) ++rank;
  }
  const float z = L.valid ? w * inv_t : -INFINITY;
  float m = seg_reduce(z, L.lane, L.end, Max());
  m = __shfl_sync(kFull, m, L.head);
  const float e = L.valid ? FEXP(z - m) : 0.f;
  float s = seg_reduce(e, L.lane, L.end, Sum());
  s = __shfl_sync(kFull, s, L.head);
  const float ph = e / s;
  float before = 0.f;   // sum of p_hat of the better-ranked candidates
  for (int j = 0; j < 32; ++j) {
    const float pj = __shfl_sync(kFull, ph, j);
    const int rj = __shfl_sync(kFull, rank, j);
    if (((L.gmask >> j) & 1u) && rj < rank) before += pj;
  }
  const bool in = on && (rank == 0 || before < top_p);
  const uint32_t inm = __ballot_sync(kFull, in);
  if (L.valid && L.lane == L.head) {
    P.nsize[L.sub] = on ? __popc(inm & L.gmask) : 0;
    if (!on) P.route[L.sub] = -1;
  }
  const int32_t gid = L.valid ? (int32_t)(P.path_base + P.slot_path[slot]) : -1;
  if (in) P.nucleus_tmp[(size_t)b * 32 + L.head + rank] = gid;
  if (on && rank == 0) {
    P.route[L.sub] = gid;
    const short4 c4 = __ldg(&P.sxy[L.sub]);
    const int x0 = c4.x, y0 = c4.y, x1 = c4.z, y1 = c4.w;
    const int ylo = min(y0, y1), yhi = max(y0, y1);
    const int mid = (int)(L.pw >> 16);
    const int X = P.X;
    auto hseg = [&](int y, int xa, int xb) { for (int x = min(xa, xb); x < max(xa, xb); ++x) atomicAdd(&P.DH[(size_t)y * X + x], 1); };
    auto vseg = [&](int x, int ya, int yb) { for (int y = min(ya, yb); y < max(ya, yb); ++y) atomicAdd(&P.DV[(size_t)y * X + x], 1); };
    auto tp = [&](int x, int y) { atomicAdd(&P.VC[(size_t)y * X + x], 1); };
    int ntp = 0;
    switch (L.shape) {
      case kStraightH: hseg(y0, x0, x1); break;
      case kStraightV: vseg(x0, y0, y1); break;
      case kHV: hseg(y0, x0, x1); vseg(x1, ylo, yhi); tp(x1, y0); ntp = 1; break;
      case kVH: vseg(x0, ylo, yhi); hseg(y1, x0, x1); tp(x0, y1); ntp = 1; break;
      case kZHVH: hseg(y0, x0, mid); vseg(mid, ylo, yhi); hseg(y1, mid, x1); tp(mid, y0); tp(mid, y1); ntp = 2; break;
      default: vseg(x0, y0, mid); hseg(mid, x0, x1); vseg(x1, mid, y1); tp(x0, mid); tp(x1, mid); ntp = 2; break;
    }
    atomicAdd(reinterpret_cast<unsigned long long*>(P.iscal),
              (unsigned long long)((x1 - x0) + abs(y1 - y0) + 2 * detour(L.pw, x0, y0, x1, y1)));
    atomicAdd(reinterpret_cast<unsigned long long*>(P.iscal + 1), (unsigned long long)ntp);
  }
}

// KI2 for the general nets' sub-nets (row f4'): a warp per sub-net of any size; the same rules
// (rank by (w desc, index asc), noise-free p_hat = softmax(w / t), nucleus = smallest prefix with
// cumulative p_hat >= top_p, route = its first) over explicit segment lists.
__global__ void __launch_bounds__(256) ki_gen_kernel(KParams P, float inv_t, float top_p) {
  const int s = blockIdx.x * 8 + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  if (s >= P.ngsub) return;
  const GSub G = P.gsub[s];
  if (!P.chosen[G.tree]) {
    if (lane == 0) { P.nsize[G.ksub] = 0; P.route[G.ksub] = -1; }
    return;
  }
  float zmax = -INFINITY;
  for (int i = lane; i < G.n; i += 32) zmax = fmaxf(zmax, P.wp[G.slot + i] * inv_t);
  zmax = warp_max_f(zmax);
  float sum = 0.f;
  for (int i = lane; i < G.n; i += 32) sum += FEXP(P.wp[G.slot + i] * inv_t - zmax);
  sum = warp_sum_f(sum);
  int cnt = 0;
  for (int b = 0; b < G.n; b += 32) {
    const int i = b + lane;
    bool in = false;
    if (i < G.n) {
      const float w = P.wp[G.slot + i];
      int rank = 0;
      float before = 0.f;   // p_hat of the better-ranked candidates
      for (int k = 0; k < G.n; ++k) {
        const float wk = P.wp[G.slot + k];
        if (wk > w || (wk == w && k < i)) { ++rank; before += FDIV(FEXP(wk * inv_t - zmax), sum); }
      }
      in = rank == 0 || before < top_p;
      const int32_t gid = (int32_t)(P.path_base + P.slot_path[G.slot + i]);
      if (in) P.nucleus_tmp[G.slot + rank] = gid;
      if (rank == 0) {
        P.route[G.ksub] = gid;
        const int X = P.X;
        int wl = 0;
        for (int q = P.gp_seg_off[G.gp + i]; q < P.gp_seg_off[G.gp + i + 1]; ++q) {
          const short4 g = P.gseg[q];
          for (int e = g.z; e < g.w; ++e)
            atomicAdd(g.x == 0 ? &P.DH[(size_t)g.y * X + e] : &P.DV[(size_t)e * X + g.y], 1);
          wl += g.w - g.z;
        }
        const int t0 = P.gp_tp_off[G.gp + i], t1 = P.gp_tp_off[G.gp + i + 1];
        for (int q = t0; q < t1; ++q) atomicAdd(&P.VC[(size_t)P.gtp[q].y * X + P.gtp[q].x], 1);
        atomicAdd(reinterpret_cast<unsigned long long*>(P.iscal), (unsigned long long)wl);
        atomicAdd(reinterpret_cast<unsigned long long*>(P.iscal + 1), (unsigned long long)(t1 - t0));
      }
    }
    cnt += __popc(__ballot_sync(kFull, in));
  }
  if (lane == 0) P.nsize[G.ksub] = cnt;
}

__global__ void __launch_bounds__(256) ki_metrics_kernel(KParams P, float beta) {
  __shared__ double sh[32];
  const int X = P.X, Y = P.Y;
  const int64_t ncell = (int64_t)X * Y;
  double tot = 0.0, cnt = 0.0, mx = 0.0;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < ncell; c += (int64_t)gridDim.x * blockDim.x) {
    const int x = (int)(c % X), y = (int)(c / X);
    if (x <= X - 2) {
      const double o = P.DH[c] + (double)beta * (P.VC[c] + P.VC[c + 1]) - (double)P.capH[c];
      if (o > 0) { tot += o; cnt += 1; mx = fmax(mx, o); }
    }
    if (y <= Y - 2) {
      const double o = P.DV[c] + (double)beta * (P.VC[c] + P.VC[c + X]) - (double)P.capVT[(size_t)x * Y + y];
      if (o > 0) { tot += o; cnt += 1; mx = fmax(mx, o); }
    }
  }
  double r;
  block_exclusive_scan(tot, sh, &r);
  if (threadIdx.x == 0) P.ipartial[3 * blockIdx.x] = r;
  block_exclusive_scan(cnt, sh, &r);
  if (threadIdx.x == 0) P.ipartial[3 * blockIdx.x + 1] = r;
  // block max
  for (int off = 16; off > 0; off >>= 1) mx = fmax(mx, __shfl_down_sync(kFull, mx, off));
  __syncthreads();
  if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = mx;
  __syncthreads();
  if (threadIdx.x == 0) {
    double m = 0.0;
    for (int i = 0; i < (int)(blockDim.x >> 5); ++i) m = fmax(m, sh[i]);
    P.ipartial[3 * blockIdx.x + 2] = m;
  }
}

__global__ void ki_finalize_kernel(KParams P, int nblocks) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  double tot = 0, cnt = 0, mx = 0;
  for (int i = 0; i < nblocks; ++i) {
    tot += P.ipartial[3 * i]; cnt += P.ipartial[3 * i + 1]; mx = fmax(mx, P.ipartial[3 * i + 2]);
  }
  P.metrics[0] = tot; P.metrics[1] = cnt; P.metrics[2] = mx;
  P.metrics[3] = (double)P.iscal[0]; P.metrics[4] = (double)P.iscal[1];
}

// ------------------------------------------------------------------------------------------
// launchers
// ------------------------------------------------------------------------------------------
static inline int cdiv(int64_t a, int64_t b) { return (int)((a + b - 1) / b); }

static int g_num_sms = 148;

size_t tile_smem_bytes() { return kBSmemBytes; }
int read_tile_prof(long long* out, int n) {   // diagnostics (DGR_DEBUG_SKIP bit 256)
  return (int)cudaMemcpyFromSymbol(out, g_tile_prof, sizeof(long long) * 8 * (size_t)(n < kProfTiles ? n : kProfTiles));
}

int prepare_kernels() {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(tile_bulk<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kBSmemBytes);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(tile_bulk<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kBSmemBytes);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(tile_bulk<true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kBSmemBytes);
  return (int)e;
}

#ifndef DGR_PDL
#define DGR_PDL 1
#endif
static cudaLaunchConfig_t pdl_config(int grid, int block, size_t smem, cudaStream_t s, cudaLaunchAttribute* attr) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  attr->id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr->val.programmaticStreamSerializationAllowed = DGR_PDL;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cfg;
}
void launch_tiles(const KParams& p, const StepArgs& a, TileMode mode, cudaStream_t s) {
  // one launch: global tiles in the first CTAs (the longest start earliest), then the pipelined tiles
  const int grid = p.ntiles + p.ntiles_slow + p.ngen_blocks;
  if (grid == 0) return;
  cudaLaunchAttribute attr;
  cudaLaunchConfig_t cfg = pdl_config(grid, kBThreads, kBSmemBytes, s, &attr);
  if (mode == kForwardOnly) cudaLaunchKernelEx(&cfg, tile_bulk<false, true>, p, a);
  else if (mode == kReverseForward) cudaLaunchKernelEx(&cfg, tile_bulk<true, true>, p, a);
  else cudaLaunchKernelEx(&cfg, tile_bulk<true, false>, p, a);
}
void launch_kg_loss(const KParams& p, const StepArgs& a, cudaStream_t s) {
  cudaLaunchAttribute attr;
  cudaLaunchConfig_t cfg = pdl_config(1, 1024, 0, s, &attr);
  cudaLaunchKernelEx(&cfg, kg_loss_kernel, p, a);
}
void launch_kg(const KParams& p, const StepArgs& a, cudaStream_t s) {
  cudaLaunchAttribute attr;
  const int nl = (p.kg_h1 - p.kg_h0) + (p.kg_v1 - p.kg_v0);
  if (nl <= 0) return;
  cudaLaunchConfig_t cfg = pdl_config(nl, kGThreads, 0, s, &attr);
  cudaLaunchKernelEx(&cfg, kg_kernel, p, a);
}
int induce_metric_blocks(const KParams& p) {
  const int64_t ncell = (int64_t)p.X * p.Y;
  const int nb = cdiv(ncell, 256);
  return nb < 1184 ? nb : 1184;
}
void launch_induce(const KParams& p, float t_final, float top_p, float /*beta*/, cudaStream_t s) {
  if (p.n_nets_l > 0) ki_tree_kernel<<<cdiv(p.n_nets_l, 256), 256, 0, s>>>(p);
  if (p.nb > 0) ki_path_kernel<<<cdiv(p.nb, 8), 256, 0, s>>>(p, 1.0f / t_final, top_p);
  if (p.ngsub > 0) ki_gen_kernel<<<cdiv(p.ngsub, 8), 256, 0, s>>>(p, 1.0f / t_final, top_p);
}
void launch_induce_metrics(const KParams& p, float beta, cudaStream_t s) {
  const int nb = induce_metric_blocks(p);
  ki_metrics_kernel<<<nb, 256, 0, s>>>(p, beta);
  ki_finalize_kernel<<<1, 32, 0, s>>>(p, nb);
}

}  // namespace dgr
