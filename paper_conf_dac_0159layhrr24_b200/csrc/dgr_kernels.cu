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
// tiles, against the whole grid in HBM.  H-type arrays are row-major in the window/grid,
// V-type arrays column-major (x-major), matching the line layouts of KG.
// ------------------------------------------------------------------------------------------
struct Win {
  int ox, oy, hs, vs;   // origin; row stride of H arrays (= width), column stride of V arrays (= height)
  __device__ __forceinline__ int h(int x, int y) const { return (y - oy) * hs + (x - ox); }
  __device__ __forceinline__ int v(int x, int y) const { return (x - ox) * vs + (y - oy); }
};

// c_i = a1 WL + a2 sqrt(L) TP + sum over the path's edges of G + beta sum over its turning points of
// the G of the incident edges; a segment's sum is S[hi] - S[lo]; path geometry from the canonical
// sub-net endpoints and the pattern word (straight, HV, VH, Z-HVH(x_m), Z-VHV(y_m)).
__device__ __forceinline__ double path_cost(const double* SH, const double* SV, const Win& W, int X, int Y,
                                            uint32_t shape, int x0, int y0, int x1, int y1, int m,
                                            const StepArgs& A) {
  const int ylo = min(y0, y1), yhi = max(y0, y1);
  // up to three segments: (is_v, line, lo, hi); inactive when lo == hi
  int v1 = 0, l1 = y0, a1 = x0, b1 = x1;
  int v2 = 0, l2 = 0, a2 = 0, b2 = 0;
  int v3 = 0, l3 = 0, a3 = 0, b3 = 0;
  int ntp = 0, tx0 = 0, ty0 = 0, tx1 = 0, ty1 = 0;
  switch (shape) {
    case kStraightH: break;
    case kStraightV: v1 = 1; l1 = x0; a1 = y0; b1 = y1; break;
    case kHV: v2 = 1; l2 = x1; a2 = ylo; b2 = yhi; ntp = 1; tx0 = x1; ty0 = y0; break;
    case kVH: v1 = 1; l1 = x0; a1 = ylo; b1 = yhi; l2 = y1; a2 = x0; b2 = x1; ntp = 1; tx0 = x0; ty0 = y1; break;
    case kZHVH:
      b1 = m; v2 = 1; l2 = m; a2 = ylo; b2 = yhi; l3 = y1; a3 = m; b3 = x1;
      ntp = 2; tx0 = m; ty0 = y0; tx1 = m; ty1 = y1; break;
    default:  // kZVHV
      v1 = 1; l1 = x0; a1 = min(y0, m); b1 = max(y0, m); l2 = m; a2 = x0; b2 = x1;
      v3 = 1; l3 = x1; a3 = min(m, y1); b3 = max(m, y1);
      ntp = 2; tx0 = x0; ty0 = m; tx1 = x1; ty1 = m; break;
  }
  auto seg = [&](int isv, int line, int lo, int hi) -> double {
    if (lo == hi) return 0.0;
    return isv ? SV[W.v(line, hi)] - SV[W.v(line, lo)] : SH[W.h(hi, line)] - SH[W.h(lo, line)];
  };
  auto tp = [&](int x, int y) -> double {
    return SH[W.h(min(x + 1, X - 1), y)] - SH[W.h(max(x - 1, 0), y)] + SV[W.v(x, min(y + 1, Y - 1))] -
           SV[W.v(x, max(y - 1, 0))];
  };
  double c = seg(v1, l1, a1, b1) + seg(v2, l2, a2, b2) + seg(v3, l3, a3, b3);
  if (ntp >= 1) c += (double)A.beta * tp(tx0, ty0);
  if (ntp >= 2) c += (double)A.beta * tp(tx1, ty1);
  c += (double)A.a_wl * (double)((x1 - x0) + (yhi - ylo)) + (double)A.a_via * (double)A.sqrt_l * ntp;
  return c;
}

// ------------------------------------------------------------------------------------------
// The tile kernel.  Shared memory (dynamic):
//   SH_s, SV_s   double[kWinMax]   S window (reverse)
//   dH_s, dV_s, VD_s int[kWinMax]  demand-event window (forward), 2^-24 fixed point
//   wst          float[kMaxBundles*32]  new logits of the tile (reverse -> forward)
//   dq_s         long long[kTreeMax]    dq_j in 2^-32 fixed point
//   q_s          float[kTreeMax]        q_j of the forward iteration
//   red_s        long long[2]           E[WL], E[TP] partial sums
// ------------------------------------------------------------------------------------------
constexpr size_t kSmemBytes = 2 * sizeof(double) * kWinMax + 3 * sizeof(int) * kWinMax +
                              sizeof(float) * kMaxBundles * 32 + sizeof(long long) * kTreeMax +
                              sizeof(float) * kTreeMax + 2 * sizeof(long long);

template <bool GLOBAL>
__device__ __forceinline__ void reverse_bundle(const KParams& P, const StepArgs& A, const TileDesc& T, int b,
                                               const double* SH, const double* SV, const Win& W,
                                               long long* dq_s, float* wst) {
  Lane L;
  lane_setup(P, b, L);
  const size_t slot = (size_t)b * 32 + L.lane;
  float w = P.wp[slot];
  const float p = group_softmax(P, A.inv_t, (uint32_t)A.k, L, w);
  const float q = L.valid ? P.q[L.tree] : 0.f;
  double c = 0.0;
  if (L.valid) {
    const short4 e = __ldg(&P.sxy[L.sub]);
    c = path_cost(SH, SV, W, P.X, P.Y, L.shape, e.x, e.y, e.z, e.w, (int)(L.pw >> 16), A);
  }
  // softmax backward dw_i = (p_i/t)(dp_i - sum_k p_k dp_k).  The weighted mean is divided by the
  // fp32 probabilities' own sum so that sum_k p_k != 1 (rounding) cannot leak c's magnitude into dw.
  const double dp = (double)q * c;
  double spd = seg_reduce((double)p * dp, L.lane, L.end, Sum());
  double sp = seg_reduce((double)p, L.lane, L.end, Sum());
  spd = __shfl_sync(kFull, spd, L.head);
  sp = __shfl_sync(kFull, sp, L.head);
  const double dw = L.valid ? (double)p * (double)A.inv_t * (dp - spd / sp) : 0.0;
  // dq_j = sum_{i in tree j} p_i c_i: reduce over this warp's lanes of each tree
  const uint32_t th = L.tm | __ballot_sync(kFull, !L.valid) | 1u;
  const uint32_t trest = th & ~L.le;
  const int tend = trest ? (__ffs(trest) - 2) : 31;
  const double pc = seg_reduce(L.valid ? (double)p * c : 0.0, L.lane, tend, Sum());
  if (L.valid && ((th >> L.lane) & 1u))
    atomicAdd(reinterpret_cast<unsigned long long*>(&dq_s[L.tree - T.tree0]),
              static_cast<unsigned long long>(__double2ll_rn(pc * kDqScale)));
  if (L.valid) {
    float m = P.mp[slot], v = P.vp[slot];
    adam_update(w, m, v, (float)dw, A);
    P.wp[slot] = w;
    P.mp[slot] = m;
    P.vp[slot] = v;
  }
  wst[(b - T.b0) * 32 + L.lane] = w;
}

// Forward events of one lane.  For a canonical sub-net (x0 < x1), s = sgn(y1 - y0), the +-pi events
// of all its candidates collapse onto 4 corner G-cells plus 2 cells per Z candidate:
//   (x0,y0): dH += A+Hs, dV += s(B+Vs)        (x1,y0): dH -= A, dV += sA, VD += A      [HV lane]
//   (x0,y1): dH += B, dV -= sB, VD += B       (x1,y1): dH -= B+Hs, dV -= s(A+Vs)       [VH lane]
//   Z-HVH(xm): (xm,y0): -pi, +s pi, +pi   (xm,y1): +pi, -s pi, +pi        [dH, dV, VD]
//   Z-VHV(ym): (x0,ym): +pi, -s pi, +pi   (x1,ym): -pi, +s pi, +pi
// with A = pi_HV, B = pi_VH, Hs = sum pi over Z-HVH, Vs = sum pi over Z-VHV.  dH is the difference
// array of the H wire demand along rows, dV along columns, VD the turning points.
template <bool GLOBAL>
__device__ __forceinline__ void forward_bundle(const KParams& P, const StepArgs& A, const TileDesc& T, int b,
                                               bool have_w, const float* wst, const float* q_s, const Win& W,
                                               int* dH_s, int* dV_s, int* VD_s, long long* red_s) {
  Lane L;
  lane_setup(P, b, L);
  const size_t slot = (size_t)b * 32 + L.lane;
  const float w = have_w ? wst[(b - T.b0) * 32 + L.lane] : P.wp[slot];
  const float p = group_softmax(P, A.inv_t, (uint32_t)A.k_next, L, w);
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
  const int Av = __shfl_sync(kFull, vq, L.head);
  const int Bv = __shfl_sync(kFull, vq, h1);
  const int S1 = __shfl_sync(kFull, sc, h1);
  const int S2 = __shfl_sync(kFull, sc, h2);
  const int Se = __shfl_sync(kFull, sc, L.end);
  int xa = 0, ya = 0, xb = 0, yb = 0;
  int ah = 0, av = 0, ad = 0, bh = 0, bv = 0, bd = 0;
  long long wl = 0, tpc = 0;
  if (L.valid) {
    const short4 e = __ldg(&P.sxy[L.sub]);
    const int x0 = e.x, y0 = e.y, x1 = e.z, y1 = e.w;
    const int s = (y1 > y0) ? 1 : -1;
    const int a = Av, bb = Bv, hs = S2 - S1, vs = Se - S2, v = vq;
    const int m = (int)(L.pw >> 16);
    int ntp = 0;
    switch (L.shape) {
      case kStraightH: xa = x0; ya = y0; ah = v; xb = x1; yb = y0; bh = -v; break;
      case kStraightV: xa = x0; ya = y0; av = v; xb = x0; yb = y1; bv = -v; break;
      case kHV:
        xa = x0; ya = y0; ah = a + hs; av = s * (bb + vs);
        xb = x1; yb = y0; bh = -a; bv = s * a; bd = a; ntp = 1; break;
      case kVH:
        xa = x0; ya = y1; ah = bb; av = -s * bb; ad = bb;
        xb = x1; yb = y1; bh = -(bb + hs); bv = -s * (a + vs); ntp = 1; break;
      case kZHVH:
        xa = m; ya = y0; ah = -v; av = s * v; ad = v;
        xb = m; yb = y1; bh = v; bv = -s * v; bd = v; ntp = 2; break;
      default:
        xa = x0; ya = m; ah = v; av = -s * v; ad = v;
        xb = x1; yb = m; bh = -v; bv = s * v; bd = v; ntp = 2; break;
    }
    wl = (long long)vq * ((x1 - x0) + abs(y1 - y0));
    tpc = (long long)vq * ntp;
  }
  if (GLOBAL) {
    const int X = P.X, Y = P.Y;
    red64(P.dH + (size_t)ya * X + xa, ah); red64(P.dVT + (size_t)xa * Y + ya, av);
    red64(P.VDH + (size_t)ya * X + xa, ad); red64(P.VDV + (size_t)xa * Y + ya, ad);
    red64(P.dH + (size_t)yb * X + xb, bh); red64(P.dVT + (size_t)xb * Y + yb, bv);
    red64(P.VDH + (size_t)yb * X + xb, bd); red64(P.VDV + (size_t)xb * Y + yb, bd);
  } else {
    if (ah) atomicAdd(&dH_s[W.h(xa, ya)], ah);
    if (av) atomicAdd(&dV_s[W.v(xa, ya)], av);
    if (ad) atomicAdd(&VD_s[W.h(xa, ya)], ad);
    if (bh) atomicAdd(&dH_s[W.h(xb, yb)], bh);
    if (bv) atomicAdd(&dV_s[W.v(xb, yb)], bv);
    if (bd) atomicAdd(&VD_s[W.h(xb, yb)], bd);
  }
  wl = seg_reduce(wl, L.lane, 31, Sum());
  tpc = seg_reduce(tpc, L.lane, 31, Sum());
  if (L.lane == 0) {
    atomicAdd(reinterpret_cast<unsigned long long*>(&red_s[0]), static_cast<unsigned long long>(wl));
    atomicAdd(reinterpret_cast<unsigned long long*>(&red_s[1]), static_cast<unsigned long long>(tpc));
  }
}

template <bool REV, bool FWD>
__global__ void __launch_bounds__(kTileThreads) tile_kernel(KParams P, StepArgs A) {
  extern __shared__ __align__(16) unsigned char smem[];
  double* SH_s = reinterpret_cast<double*>(smem);
  double* SV_s = SH_s + kWinMax;
  int* dH_s = reinterpret_cast<int*>(SV_s + kWinMax);
  int* dV_s = dH_s + kWinMax;
  int* VD_s = dV_s + kWinMax;
  float* wst = reinterpret_cast<float*>(VD_s + kWinMax);
  long long* dq_s = reinterpret_cast<long long*>(wst + kMaxBundles * 32);
  float* q_s = reinterpret_cast<float*>(dq_s + kTreeMax);
  long long* red_s = reinterpret_cast<long long*>(q_s + kTreeMax);

  const TileDesc T = P.tiles[blockIdx.x];
  const int tid = threadIdx.x, warp = tid >> 5, nwarp = kTileThreads / 32;
  const int ncell = T.ww * T.wh;
  const int X = P.X, Y = P.Y;
  const Win Wg{0, 0, X, Y};
  const Win Ws{T.wx0, T.wy0, T.ww, T.wh};

  // ---------------- reverse of iteration k ----------------
  if (REV) {
    if (!T.global) {
      for (int i = tid; i < ncell; i += kTileThreads) {
        const int yi = i / T.ww, xi = i - yi * T.ww;
        SH_s[i] = P.SH[(size_t)(T.wy0 + yi) * X + T.wx0 + xi];
      }
      for (int i = tid; i < ncell; i += kTileThreads) {
        const int xi = i / T.wh, yi = i - xi * T.wh;
        SV_s[i] = P.SVT[(size_t)(T.wx0 + xi) * Y + T.wy0 + yi];
      }
    }
    for (int i = tid; i < T.ntree; i += kTileThreads) dq_s[i] = 0;
    __syncthreads();
    for (int b = T.b0 + warp; b < T.b0 + T.nb; b += nwarp) {
      if (T.global) reverse_bundle<true>(P, A, T, b, P.SH, P.SVT, Wg, dq_s, wst);
      else reverse_bundle<false>(P, A, T, b, SH_s, SV_s, Ws, dq_s, wst);
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
        const double qj = (double)P.q[j];
        sq += qj * ((double)dq_s[j - T.tree0] * kDqInv);
        sw += qj;
      }
      sq /= sw;
      for (int j = a; j < b; ++j) {
        const double du = (b - a == 1) ? 0.0
                                       : (double)P.q[j] * (double)A.inv_t * ((double)dq_s[j - T.tree0] * kDqInv - sq);
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
      for (int i = tid; i < ncell; i += kTileThreads) { dH_s[i] = 0; dV_s[i] = 0; VD_s[i] = 0; }
    if (tid < 2) red_s[tid] = 0;
    __syncthreads();
    for (int b = T.b0 + warp; b < T.b0 + T.nb; b += nwarp) {
      if (T.global) forward_bundle<true>(P, A, T, b, REV, wst, q_s, Wg, dH_s, dV_s, VD_s, red_s);
      else forward_bundle<false>(P, A, T, b, REV, wst, q_s, Ws, dH_s, dV_s, VD_s, red_s);
    }
    __syncthreads();
    if (!T.global) {
      // flush the window once: row-major fields along rows, column-major fields along columns
      for (int i = tid; i < ncell; i += kTileThreads) {
        const int yi = i / T.ww, xi = i - yi * T.ww;
        const size_t g = (size_t)(T.wy0 + yi) * X + T.wx0 + xi;
        red64(P.dH + g, dH_s[i]);
        red64(P.VDH + g, VD_s[i]);
      }
      for (int i = tid; i < ncell; i += kTileThreads) {
        const int xi = i / T.wh, yi = i - xi * T.wh;
        const size_t g = (size_t)(T.wx0 + xi) * Y + T.wy0 + yi;
        red64(P.dVT + g, dV_s[i]);
        red64(P.VDV + g, VD_s[yi * T.ww + xi]);
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
