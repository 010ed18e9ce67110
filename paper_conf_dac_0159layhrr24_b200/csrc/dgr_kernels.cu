// dgr_kernels.cu — sm_100a kernels of the DGR solver iteration (§4.3-4.5).
//
// One iteration k is two kernels (plus the NCCL allreduce of the demand when world > 1):
//
//   KG   per G-cell line (CTA / line): scan of the difference arrays -> demand d (Eq. (10),
//        P:556-564), overflow cost f(cap - d) (Eq. (9)), gradient map G = -a3 f'(cap - d), and
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

#include "dgr_internal.h"

namespace dgr {

constexpr unsigned kFull = 0xffffffffu;

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

__device__ __forceinline__ float gumbel(uint64_t seed, uint64_t idx, uint32_t k, uint32_t stream) {
  const uint4 r = philox4x32_10(make_uint4((uint32_t)(idx >> 2), (uint32_t)(idx >> 34), k, stream),
                                make_uint2((uint32_t)seed, (uint32_t)(seed >> 32)));
  const uint32_t s = (uint32_t)idx & 3u;
  const uint32_t w = s == 0 ? r.x : (s == 1 ? r.y : (s == 2 ? r.z : r.w));
  const float u = ((float)(w >> 9) + 0.5f) * (1.0f / 8388608.0f);
  return -logf(-logf(u));
}

// ------------------------------------------------------------------------------------------
// Per-lane view of a bundle: which sub-net group / tree / global candidate this lane is.
// ------------------------------------------------------------------------------------------
struct Lane {
  int lane, head, end;
  uint32_t pw, shape, le, gmask, hm, tm;
  bool valid;
  int sub, tree;
  int64_t gid, lpath;
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
  L.tree = bi.z + __popc(L.tm & L.le & ~1u);
  L.lpath = (int64_t)bi.x + L.lane;
  L.gid = P.path_base + L.lpath;
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

// p_i = softmax over the sub-net group of (w_i + g_i) / t (reading Q1)
__device__ __forceinline__ float group_softmax(const KParams& P, float inv_t, uint32_t k, const Lane& L, float w) {
  const float z = L.valid ? (w + gumbel(P.seed, (uint64_t)L.gid, k, 0u)) * inv_t : -INFINITY;
  float m = seg_reduce(z, L.lane, L.end, Max());
  m = __shfl_sync(kFull, m, L.head);
  const float e = L.valid ? __expf(z - m) : 0.f;
  float s = seg_reduce(e, L.lane, L.end, Sum());
  s = __shfl_sync(kFull, s, L.head);
  return L.valid ? e / s : 0.f;
}

__device__ __forceinline__ void red64(long long* p, long long v) {
  if (v != 0) atomicAdd(reinterpret_cast<unsigned long long*>(p), static_cast<unsigned long long>(v));
}

__device__ __forceinline__ void adam_update(float& w, float& m, float& v, float g, const StepArgs& A) {
  m = fmaf(0.1f, g - m, m);                         // m.lerp_(g, 1 - beta1)
  v = fmaf(0.999f, v, 0.001f * g * g);              // v * beta2 + (1 - beta2) g^2
  const float denom = sqrtf(v) * A.inv_sqrt_bc2 + 1e-8f;
  w -= A.lr_over_bc1 * (m / denom);
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

struct Shape6 {
  bool sh, sv, hv, vh, zh, zv;
  __device__ __forceinline__ explicit Shape6(uint32_t s)
      : sh(s == kStraightH), sv(s == kStraightV), hv(s == kHV), vh(s == kVH), zh(s == kZHVH), zv(s == kZVHV) {}
};

// c_i = a1 WL + a2 sqrt(L) TP + sum over the path's edges of G + beta sum over its turning points of
// the G of the incident edges; a segment's sum is S[hi] - S[lo].  Branch-free: the pattern selects
// up to three segments and two turning points (straight, HV, VH, Z-HVH(x_m), Z-VHV(y_m)); unused
// slots read valid cells and are weighted by 0.
__device__ __forceinline__ double path_cost(const double* S, const Win& W, int X, int Y, uint32_t shape, int x0,
                                            int y0, int x1, int y1, int m, const StepArgs& A) {
  const Shape6 k(shape);
  const int ylo = min(y0, y1), yhi = max(y0, y1);
  // segment 1 (always)
  const bool v1 = k.sv | k.vh | k.zv;
  const int l1 = v1 ? x0 : y0;
  const int a1 = v1 ? (k.zv ? min(y0, m) : ylo) : x0;
  const int b1 = v1 ? (k.zv ? max(y0, m) : yhi) : (k.zh ? m : x1);
  // segment 2 (L and Z)
  const bool v2 = k.hv | k.zh;
  const int l2 = k.hv ? x1 : (k.vh ? y1 : m);
  const int a2 = v2 ? ylo : x0;
  const int b2 = v2 ? yhi : x1;
  // segment 3 (Z)
  const int l3 = k.zh ? y1 : x1;
  const int a3 = k.zh ? m : min(m, y1);
  const int b3 = k.zh ? x1 : max(m, y1);
  const bool s2 = !(k.sh | k.sv), s3 = k.zh | k.zv;
  // turning points (default cell (x0, y0) when unused)
  const int tx0 = k.hv ? x1 : (k.zh ? m : x0);
  const int ty0 = k.hv ? y0 : (k.vh ? y1 : (k.zv ? m : y0));
  const int tx1 = k.zh ? m : (k.zv ? x1 : x0);
  const int ty1 = k.zh ? y1 : (k.zv ? m : y0);
  const int ntp = (k.hv | k.vh) ? 1 : (s3 ? 2 : 0);
  auto sidx = [&](bool isv, int line, int pos) { return isv ? W.v(line, pos) : W.h(pos, line); };
  const int i1b = sidx(v1, l1, b1), i1a = sidx(v1, l1, a1);
  const int i2b = s2 ? sidx(v2, l2, b2) : i1b, i2a = s2 ? sidx(v2, l2, a2) : i1b;
  const int i3b = s3 ? sidx(k.zv, l3, b3) : i1b, i3a = s3 ? sidx(k.zv, l3, a3) : i1b;
  const double seg = (S[i1b] - S[i1a]) + (S[i2b] - S[i2a]) + (S[i3b] - S[i3a]);
  auto tp = [&](int x, int y) -> double {
    return S[W.h(min(x + 1, X - 1), y)] - S[W.h(max(x - 1, 0), y)] + S[W.v(x, min(y + 1, Y - 1))] -
           S[W.v(x, max(y - 1, 0))];
  };
  const double t0 = tp(tx0, ty0), t1 = tp(tx1, ty1);
  const double tps = (ntp >= 1 ? t0 : 0.0) + (ntp >= 2 ? t1 : 0.0);
  return seg + (double)A.beta * tps + (double)A.a_wl * (double)((x1 - x0) + (yhi - ylo)) +
         (double)A.a_via * (double)A.sqrt_l * ntp;
}

__device__ __forceinline__ void red_shared_add(uint32_t saddr, int v) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.s32 p, %1, 0;\n\t@p red.shared.add.s32 [%0], %1;\n\t}" ::"r"(saddr), "r"(v)
               : "memory");
}

// g = -ln(-ln u) from one Philox word
__device__ __forceinline__ float gumbel_word(uint32_t w) {
  const float u = ((float)(w >> 9) + 0.5f) * (1.0f / 8388608.0f);
  return -logf(-logf(u));
}

// Gumbel noise of a warp's contiguous candidates gid0 .. gid0+n-1 into g[0..n): one Philox4x32-10
// call per 4 consecutive candidates (counter gid >> 2), spread over the lanes.
__device__ __forceinline__ void warp_noise(float* g, uint64_t seed, int64_t gid0, int n, uint32_t k, int lane) {
  const int64_t c0 = gid0 >> 2, c1 = (gid0 + n - 1) >> 2;
  const uint2 key = make_uint2((uint32_t)seed, (uint32_t)(seed >> 32));
  for (int64_t c = c0 + lane; c <= c1; c += 32) {
    const uint4 r = philox4x32_10(make_uint4((uint32_t)c, (uint32_t)(c >> 32), k, 0u), key);
    const int64_t i0 = c * 4 - gid0;
    if (i0 >= 0 && i0 < n) g[i0] = gumbel_word(r.x);
    if (i0 + 1 >= 0 && i0 + 1 < n) g[i0 + 1] = gumbel_word(r.y);
    if (i0 + 2 >= 0 && i0 + 2 < n) g[i0 + 2] = gumbel_word(r.z);
    if (i0 + 3 >= 0 && i0 + 3 < n) g[i0 + 3] = gumbel_word(r.w);
  }
  __syncwarp();
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
  L.tree = bi.z + __popc(L.tm & L.le & ~1u);
  L.lpath = (int64_t)bi.x + L.lane;
  L.gid = P.path_base + L.lpath;
}

__device__ __forceinline__ float softmax_from_noise(const Lane& L, float w, float g, float inv_t) {
  const float z = L.valid ? (w + g) * inv_t : -INFINITY;
  float m = seg_reduce(z, L.lane, L.end, Max());
  m = __shfl_sync(kFull, m, L.head);
  const float e = L.valid ? __expf(z - m) : 0.f;
  float s = seg_reduce(e, L.lane, L.end, Sum());
  s = __shfl_sync(kFull, s, L.head);
  return L.valid ? __fdividef(e, s) : 0.f;
}

// ------------------------------------------------------------------------------------------
// The tile kernel.  Shared memory (dynamic), region A is reused between the two halves:
//   A, reverse:  S_s   double[2 kWinMax]          S window: H part, then V part
//   A, forward:  ev_s  int[3 kWinMax]             demand-event window dH | dV | VD, 2^-24 fixed point
//                g_s   float[kWarps][kWarpCand]   Gumbel noise of each warp's candidates
//   wst    float[kMaxBundles * 32]    new logits of the tile (reverse -> forward)
//   dq_s   long long[kTreeMax]        dq_j in 2^-32 fixed point
//   q_s    float[kTreeMax]            q_j (iteration k in the reverse, k_next in the forward)
//   red_s  long long[2]               E[WL], E[TP] partial sums
// Each warp owns a contiguous range of the tile's bundles, so its candidates are contiguous.
// ------------------------------------------------------------------------------------------
constexpr int kWarps = kTileThreads / 32;
constexpr int kWarpBundles = (kMaxBundles + kWarps - 1) / kWarps;
constexpr int kWarpCand = kWarpBundles * 32;
constexpr size_t kRegionA = 2 * sizeof(double) * kWinMax;
static_assert(3 * sizeof(int) * kWinMax + sizeof(float) * kWarps * kWarpCand <= kRegionA, "region A too small");
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
  float w = P.wp[slot], m = P.mp[slot], v = P.vp[slot], p = P.pp[slot];
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
      wn = P.wp[slot + 32]; mn = P.mp[slot + 32]; vn = P.vp[slot + 32]; pn = P.pp[slot + 32];
      if (b + 2 < bw1) { bi1 = __ldg(&P.binfo[b + 2]); pw1 = __ldg(&P.pword[slot + 64]); }
    }
    const float q = L.valid ? q_s[L.tree - T.tree0] : 0.f;
    const double c = L.valid ? path_cost(S, W, P.X, P.Y, L.shape, e.x, e.y, e.z, e.w, (int)(L.pw >> 16), A) : 0.0;
    // softmax backward dw_i = (p_i/t)(dp_i - sum_k p_k dp_k / sum_k p_k): differences to the group
    // head's dp are formed in fp64 and reduced in fp32, so neither the magnitude of c nor
    // sum_k p_k != 1 (rounding) leaks into dw.
    const double dp = (double)q * c;
    const double dref = __shfl_sync(kFull, dp, L.head);
    const float dd = (float)(dp - dref);
    float sa = seg_reduce(p * dd, L.lane, L.end, Sum());
    float sb = seg_reduce(p, L.lane, L.end, Sum());
    sa = __shfl_sync(kFull, sa, L.head);
    sb = __shfl_sync(kFull, sb, L.head);
    const float dw = L.valid ? p * A.inv_t * (dd - __fdividef(sa, sb)) : 0.f;
    // dq_j = sum_{i in tree j} p_i c_i: reduce over this warp's lanes of each tree (fp64: the tree
    // gradient is a difference of such sums)
    const uint32_t th = L.tm | __ballot_sync(kFull, !L.valid) | 1u;
    const uint32_t trest = th & ~L.le;
    const int tend = trest ? (__ffs(trest) - 2) : 31;
    const double pc = seg_reduce(L.valid ? (double)p * c : 0.0, L.lane, tend, Sum());
    if (L.valid && ((th >> L.lane) & 1u))
      atomicAdd(reinterpret_cast<unsigned long long*>(&dq_s[L.tree - T.tree0]),
                static_cast<unsigned long long>(__double2ll_rn(pc * kDqScale)));
    if (L.valid) {
      adam_update(w, m, v, dw, A);
      P.wp[slot] = w;
      P.mp[slot] = m;
      P.vp[slot] = v;
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
template <bool GLOBAL>
__device__ __forceinline__ void forward_warp(const KParams& P, const StepArgs& A, const TileDesc& T, int bw0,
                                             int bw1, bool have_w, const float* wst, const float* q_s, float* g_s,
                                             const Win& W, int* ev_s, long long* red_s) {
  const int lane = threadIdx.x & 31;
  const int4 bfirst = __ldg(&P.binfo[bw0]);
  const int4 blast = __ldg(&P.binfo[bw1 - 1]);
  warp_noise(g_s, P.seed, P.path_base + bfirst.x, blast.x + blast.w - bfirst.x, (uint32_t)A.k_next, lane);
  const uint32_t ev_base = (uint32_t)__cvta_generic_to_shared(ev_s);
  long long wl = 0, tpc = 0;
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
    const float g = L.valid ? g_s[L.lpath - bfirst.x] : 0.f;
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
    const int nh = __popc(__ballot_sync(kFull, L.shape == kZHVH) & L.gmask);
    const int h1 = min(L.head + 1, 31), h2 = min(L.head + 1 + nh, 31);
    const int a = __shfl_sync(kFull, vq, L.head);
    const int bb = __shfl_sync(kFull, vq, h1);
    const int S1 = __shfl_sync(kFull, sc, h1);
    const int S2 = __shfl_sync(kFull, sc, h2);
    const int Se = __shfl_sync(kFull, sc, L.end);
    const int x0 = e.x, y0 = e.y, x1 = e.z, y1 = e.w;
    const int s = (y1 > y0) ? 1 : -1;
    const int hs = S2 - S1, vs = Se - S2, v = vq;
    const int mm = (int)(L.pw >> 16);
    const int fSH = L.shape == kStraightH, fSV = L.shape == kStraightV, fHV = L.shape == kHV;
    const int fVH = L.shape == kVH, fZH = L.shape == kZHVH, fZV = L.shape == kZVHV;
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
        red64(P.dH + (size_t)ya * X + xa, ah); red64(P.dVT + (size_t)xa * Y + ya, av);
        red64(P.VDH + (size_t)ya * X + xa, ad); red64(P.VDV + (size_t)xa * Y + ya, ad);
        red64(P.dH + (size_t)yb * X + xb, bh); red64(P.dVT + (size_t)xb * Y + yb, bv);
        red64(P.VDH + (size_t)yb * X + xb, bd); red64(P.VDV + (size_t)xb * Y + yb, bd);
      }
      const int ntp = fHV + fVH + 2 * fZ;
      wl += (long long)vq * ((x1 - x0) + abs(y1 - y0));
      tpc += (long long)vq * ntp;
    }
    if (!GLOBAL) {
      const int hv2 = 2 * W.hv;   // VD part of the event window
      const int ia_h = W.h(xa, ya), ib_h = W.h(xb, yb);
      red_shared_add(ev_base + 4u * ia_h, ah);
      red_shared_add(ev_base + 4u * W.v(xa, ya), av);
      red_shared_add(ev_base + 4u * (hv2 + ia_h), ad);
      red_shared_add(ev_base + 4u * ib_h, bh);
      red_shared_add(ev_base + 4u * W.v(xb, yb), bv);
      red_shared_add(ev_base + 4u * (hv2 + ib_h), bd);
    }
    L = Ln; e = en;
    slot += 32;
  }
  wl = seg_reduce(wl, lane, 31, Sum());
  tpc = seg_reduce(tpc, lane, 31, Sum());
  if (lane == 0) {
    atomicAdd(reinterpret_cast<unsigned long long*>(&red_s[0]), static_cast<unsigned long long>(wl));
    atomicAdd(reinterpret_cast<unsigned long long*>(&red_s[1]), static_cast<unsigned long long>(tpc));
  }
}

template <bool REV, bool FWD>
__global__ void __launch_bounds__(kTileThreads, 3) tile_kernel(KParams P, StepArgs A) {
  extern __shared__ __align__(16) unsigned char smem[];
  double* S_s = reinterpret_cast<double*>(smem);                 // region A (reverse)
  int* ev_s = reinterpret_cast<int*>(smem);                      // region A (forward)
  float* g_all = reinterpret_cast<float*>(ev_s + 3 * kWinMax);   // region A (forward)
  float* wst = reinterpret_cast<float*>(smem + kRegionA);
  long long* dq_s = reinterpret_cast<long long*>(wst + kMaxBundles * 32);
  float* q_s = reinterpret_cast<float*>(dq_s + kTreeMax);
  long long* red_s = reinterpret_cast<long long*>(q_s + kTreeMax);

  const TileDesc T = P.tiles[blockIdx.x];
  const int tid = threadIdx.x, warp = tid >> 5;
  const int ncell = T.ww * T.wh;
  const int X = P.X, Y = P.Y;
  const Win Wg{0, 0, X, Y, X * Y};
  const Win Ws{T.wx0, T.wy0, T.ww, T.wh, ncell};
  float* g_s = g_all + warp * kWarpCand;
  // this warp's contiguous bundle range
  const int per = (T.nb + kWarps - 1) / kWarps;
  const int bw0 = T.b0 + min(warp * per, T.nb), bw1 = T.b0 + min((warp + 1) * per, T.nb);

  // ---------------- reverse of iteration k ----------------
  if (REV) {
    if (!T.global) {
      for (int i = tid; i < ncell; i += kTileThreads) {
        const int yi = i / T.ww, xi = i - yi * T.ww;
        S_s[i] = P.SH[(size_t)(T.wy0 + yi) * X + T.wx0 + xi];
      }
      for (int i = tid; i < ncell; i += kTileThreads) {
        const int xi = i / T.wh, yi = i - xi * T.wh;
        S_s[ncell + i] = P.SVT[(size_t)(T.wx0 + xi) * Y + T.wy0 + yi];
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
          const float z = (P.wt[j] + gumbel(P.seed, (uint64_t)(P.tree_base + j), (uint32_t)A.k_next, 1u)) * A.inv_t;
          q_s[j - T.tree0] = z;
          zmax = fmaxf(zmax, z);
        }
        float s = 0.f;
        for (int j = a; j < b; ++j) { const float e = __expf(q_s[j - T.tree0] - zmax); q_s[j - T.tree0] = e; s += e; }
        const float inv = 1.f / s;
        for (int j = a; j < b; ++j) { q_s[j - T.tree0] *= inv; P.q[j] = q_s[j - T.tree0]; }
      }
    }
  }

  // ---------------- forward of iteration k_next ----------------
  if (FWD) {
    if (!T.global)
      for (int i = tid; i < 3 * ncell; i += kTileThreads) ev_s[i] = 0;
    if (tid < 2) red_s[tid] = 0;
    __syncthreads();
    if (bw0 < bw1) {
      if (T.global) forward_warp<true>(P, A, T, bw0, bw1, REV, wst, q_s, g_s, Wg, ev_s, red_s);
      else forward_warp<false>(P, A, T, bw0, bw1, REV, wst, q_s, g_s, Ws, ev_s, red_s);
    }
    __syncthreads();
    if (!T.global) {
      // flush the window once: row-major fields along rows, column-major fields along columns
      for (int i = tid; i < ncell; i += kTileThreads) {
        const int yi = i / T.ww, xi = i - yi * T.ww;
        const size_t g = (size_t)(T.wy0 + yi) * X + T.wx0 + xi;
        red64(P.dH + g, ev_s[i]);
        red64(P.VDH + g, ev_s[2 * ncell + i]);
      }
      for (int i = tid; i < ncell; i += kTileThreads) {
        const int xi = i / T.wh, yi = i - xi * T.wh;
        const size_t g = (size_t)(T.wx0 + xi) * Y + T.wy0 + yi;
        red64(P.dVT + g, ev_s[ncell + i]);
        red64(P.VDV + g, ev_s[2 * ncell + yi * T.ww + xi]);
      }
    }
    if (tid == 0) { red64(P.scal, red_s[0]); red64(P.scal + 1, red_s[1]); }
  }
}

// ------------------------------------------------------------------------------------------
// KG: one CTA per line (Y H-rows, then X V-columns).  Scan of the difference array gives the
// wire demand W; d = (W + beta (VD_a + VD_b)) 2^-24 (Eq. (10), reading Q3); overflow cost
// f(cap - d) (Eq. (9)); G = dcost/dd = -a3 f'(cap - d); S = exclusive prefix of G (fp64).
// The line's difference and turning-point entries are cleared for the next forward.
// ------------------------------------------------------------------------------------------
constexpr int kGThreads = 256;
constexpr int kGItems = 8;

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

__global__ void __launch_bounds__(kGThreads) kg_kernel(KParams P, StepArgs A) {
  __shared__ long long shl[32];
  __shared__ double shd[32];
  const int line = blockIdx.x;
  const bool isH = line < P.Y;
  const int n = isH ? P.X : P.Y;
  const int ln = isH ? line : line - P.Y;
  const size_t base = (size_t)ln * n;
  long long* diff = (isH ? P.dH : P.dVT) + base;
  long long* vd = (isH ? P.VDH : P.VDV) + base;
  const float* cap = (isH ? P.capH : P.capVT) + base;
  double* S = (isH ? P.SH : P.SVT) + base;
  float* dout = (isH ? P.dOutH : P.dOutVT) + base;
  const double beta = A.beta;
  long long carryW = 0;
  double carryS = 0.0, of = 0.0;
  for (int c0 = 0; c0 < n; c0 += kGThreads * kGItems) {
    const int pos0 = c0 + threadIdx.x * kGItems;
    long long v[kGItems], t[kGItems + 1];
#pragma unroll
    for (int i = 0; i < kGItems; ++i) {
      v[i] = (pos0 + i < n) ? diff[pos0 + i] : 0;
      t[i] = (pos0 + i < n) ? vd[pos0 + i] : 0;
    }
    t[kGItems] = (pos0 + kGItems < n) ? vd[pos0 + kGItems] : 0;
    long long run = 0;
#pragma unroll
    for (int i = 0; i < kGItems; ++i) { run += v[i]; v[i] = run; }   // local inclusive
    long long totW;
    const long long offW = block_exclusive_scan(run, shl, &totW);   // (synchronises: all reads done)
#pragma unroll
    for (int i = 0; i < kGItems; ++i)
      if (pos0 + i < n) { diff[pos0 + i] = 0; vd[pos0 + i] = 0; }
    double g[kGItems];
    double grun = 0.0;
#pragma unroll
    for (int i = 0; i < kGItems; ++i) {
      const int pos = pos0 + i;
      double G = 0.0;
      if (pos < n - 1) {
        const long long W = carryW + offW + v[i];
        const double d = (double)W * kFixInv + beta * ((double)(t[i] + t[i + 1]) * kFixInv);
        const double r = (double)cap[pos] - d;
        if (A.f_kind == 0) {
          // sigmoid: f(r) = 1/(1+exp(s r)) = sigma(-s r); -f'(r) = s sigma(s r) sigma(-s r).
          // fp64 here (one exp per edge): G feeds every candidate's cost difference.
          const double sr = (double)A.f_slope * r;
          const double e = exp(-fabs(sr));
          const double inv = 1.0 / (1.0 + e);
          of += (sr > 0.0) ? e * inv : inv;
          G = (double)A.a_of * (double)A.f_slope * e * inv * inv;
        } else {
          of += r < 0.0 ? -r : 0.0;
          G = (d > (double)cap[pos]) ? (double)A.a_of : 0.0;
        }
        if (A.store_d) dout[pos] = (float)d;
      } else if (pos == n - 1 && A.store_d) {
        dout[pos] = 0.f;
      }
      g[i] = grun;          // local exclusive
      grun += G;
    }
    double totS;
    const double offS = block_exclusive_scan(grun, shd, &totS);
#pragma unroll
    for (int i = 0; i < kGItems; ++i) {
      const int pos = pos0 + i;
      if (pos < n) S[pos] = carryS + offS + g[i];
    }
    carryW += totW;
    carryS += totS;
  }
  // deterministic block reduction of the overflow cost
  double tot;
  block_exclusive_scan(of, shd, &tot);
  if (threadIdx.x == 0) P.partial[line] = tot;
}

__global__ void __launch_bounds__(256) kg_finalize_kernel(KParams P, StepArgs A) {
  __shared__ double sh[32];
  const int nl = P.X + P.Y;
  double s = 0.0;
  for (int i = threadIdx.x; i < nl; i += blockDim.x) s += P.partial[i];
  double tot;
  block_exclusive_scan(s, sh, &tot);
  if (threadIdx.x == 0) {
    const double ewl = (double)P.scal[0] * kFixInv;
    const double etp = (double)P.scal[1] * kFixInv;
    const double via = (double)A.sqrt_l * etp;
    P.loss[0] = (double)A.a_wl * ewl + (double)A.a_via * via + (double)A.a_of * tot;
    P.loss[1] = ewl;
    P.loss[2] = via;
    P.loss[3] = tot;
    P.scal[0] = 0;
    P.scal[1] = 0;
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
  P.tree_choice[n] = (int32_t)(P.tree_base + best);
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
  const float e = L.valid ? __expf(z - m) : 0.f;
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
  if (in) P.nucleus_tmp[(size_t)(L.lpath - (L.lane - L.head)) + rank] = (int32_t)L.gid;
  if (on && rank == 0) {
    P.route[L.sub] = (int32_t)L.gid;
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
    atomicAdd(reinterpret_cast<unsigned long long*>(P.iscal), (unsigned long long)((x1 - x0) + abs(y1 - y0)));
    atomicAdd(reinterpret_cast<unsigned long long*>(P.iscal + 1), (unsigned long long)ntp);
  }
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

size_t tile_smem_bytes() { return kSmemBytes; }

int prepare_kernels() {
  cudaError_t e = cudaFuncSetAttribute(tile_kernel<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemBytes);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(tile_kernel<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemBytes);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(tile_kernel<true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemBytes);
  return (int)e;
}

void launch_tiles(const KParams& p, const StepArgs& a, TileMode mode, cudaStream_t s) {
  if (p.ntiles <= 0) return;
  if (mode == kForwardOnly) tile_kernel<false, true><<<p.ntiles, kTileThreads, kSmemBytes, s>>>(p, a);
  else if (mode == kReverseForward) tile_kernel<true, true><<<p.ntiles, kTileThreads, kSmemBytes, s>>>(p, a);
  else tile_kernel<true, false><<<p.ntiles, kTileThreads, kSmemBytes, s>>>(p, a);
}
void launch_kg(const KParams& p, const StepArgs& a, cudaStream_t s) {
  kg_kernel<<<p.X + p.Y, kGThreads, 0, s>>>(p, a);
  kg_finalize_kernel<<<1, 256, 0, s>>>(p, a);
}
int induce_metric_blocks(const KParams& p) {
  const int64_t ncell = (int64_t)p.X * p.Y;
  const int nb = cdiv(ncell, 256);
  return nb < 1184 ? nb : 1184;
}
void launch_induce(const KParams& p, float t_final, float top_p, float /*beta*/, cudaStream_t s) {
  if (p.n_nets_l > 0) ki_tree_kernel<<<cdiv(p.n_nets_l, 256), 256, 0, s>>>(p);
  if (p.nb > 0) ki_path_kernel<<<cdiv(p.nb, 8), 256, 0, s>>>(p, 1.0f / t_final, top_p);
}
void launch_induce_metrics(const KParams& p, float beta, cudaStream_t s) {
  const int nb = induce_metric_blocks(p);
  ki_metrics_kernel<<<nb, 256, 0, s>>>(p, beta);
  ki_finalize_kernel<<<1, 32, 0, s>>>(p, nb);
}

}  // namespace dgr
