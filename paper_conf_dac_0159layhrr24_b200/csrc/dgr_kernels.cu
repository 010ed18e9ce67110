// dgr_kernels.cu — sm_100a kernels of one DGR solver iteration (§4.3-4.5).
//
//   KQ  tree-level Gumbel-softmax q_j                     §4.4 P:827-829          (thread / net)
//   KF  path-level Gumbel-softmax p_i, pi_i = q p_i and the expected-demand scatter of Eq. (10)
//        as +-pi events at segment ends into per-line difference arrays and a
//       per-G-cell turning-point array; E[WL], E[TP] of Eqs. (11)/(12)          (warp / bundle)
//   KG  per line: scan -> demand d, overflow cost f(cap - d) of Eq. (9), gradient map
//       G = -a3 f'(cap - d), exclusive prefix S of G along the line             (CTA / line)
//   KB  reverse: c_i = dcost/dpi_i from O(1) S differences per segment and turning point,
//       softmax backward over the sub-net group, dq accumulation, fused Adam   (warp / bundle)
//   KT  tree-level softmax backward + Adam                                       (thread / net)
//   KI* discrete induction of §4.5
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
__device__ __forceinline__ float group_softmax(const KParams& P, const StepArgs& A, const Lane& L, float w) {
  const float z = L.valid ? (w + gumbel(P.seed, (uint64_t)L.gid, (uint32_t)A.k, 0u)) * A.inv_t : -INFINITY;
  float m = seg_reduce(z, L.lane, L.end, Max());
  m = __shfl_sync(kFull, m, L.head);
  const float e = L.valid ? __expf(z - m) : 0.f;
  float s = seg_reduce(e, L.lane, L.end, Sum());
  s = __shfl_sync(kFull, s, L.head);
  return L.valid ? e / s : 0.f;
}

// ------------------------------------------------------------------------------------------
// KQ: q_j = softmax over the net's trees of (w_j + g_j)/t (stream 1)
// ------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) kq_kernel(KParams P, StepArgs A) {
  const int n = blockIdx.x * blockDim.x + threadIdx.x;
  if (n >= P.n_nets_l) return;
  const int a = P.net_tree_off[n], b = P.net_tree_off[n + 1];
  if (b - a == 1) { P.q[a] = 1.f; return; }
  float zmax = -INFINITY;
  for (int j = a; j < b; ++j) {
    const float z = (P.wt[j] + gumbel(P.seed, (uint64_t)(P.tree_base + j), (uint32_t)A.k, 1u)) * A.inv_t;
    P.q[j] = z;
    zmax = fmaxf(zmax, z);
  }
  float s = 0.f;
  for (int j = a; j < b; ++j) { const float e = __expf(P.q[j] - zmax); P.q[j] = e; s += e; }
  const float inv = 1.f / s;
  for (int j = a; j < b; ++j) P.q[j] *= inv;
}

// ------------------------------------------------------------------------------------------
// KF: forward scatter.  For a canonical sub-net (x0 < x1) with sign s = sgn(y1 - y0) the +-pi
// events of all its candidates collapse onto 4 corner G-cells plus 2 cells per Z candidate:
//   (x0,y0): dH += A+Hs, dV += s(B+Vs)        (x1,y0): dH -= A, dV += sA, VD += A
//   (x0,y1): dH += B, dV -= sB, VD += B       (x1,y1): dH -= B+Hs, dV -= s(A+Vs)
//   Z-HVH(xm): (xm,y0): -pi, +s pi, +pi   (xm,y1): +pi, -s pi, +pi        [dH, dV, VD]
//   Z-VHV(ym): (x0,ym): +pi, -s pi, +pi   (x1,ym): -pi, +s pi, +pi
// where A = pi_HV, B = pi_VH, Hs = sum pi over Z-HVH, Vs = sum pi over Z-VHV.  dH is the
// difference array of the H wire demand along rows, dV along columns, VD the turning points.
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ void red64(long long* p, long long v) {
  if (v != 0) atomicAdd(reinterpret_cast<unsigned long long*>(p), static_cast<unsigned long long>(v));
}
__device__ __forceinline__ void add_cell(const KParams& P, int x, int y, long long dh, long long dv, long long vd) {
  red64(P.dH + (size_t)y * P.X + x, dh);
  red64(P.dVT + (size_t)x * P.Y + y, dv);
  red64(P.VD + (size_t)y * P.X + x, vd);
}

__global__ void __launch_bounds__(256) kf_kernel(KParams P, StepArgs A) {
  const int b = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (b >= P.nb) return;
  Lane L;
  lane_setup(P, b, L);
  const size_t slot = (size_t)b * 32 + L.lane;
  const float w = P.wp[slot];
  const float p = group_softmax(P, A, L, w);
  const float q = L.valid ? __ldg(&P.q[L.tree]) : 0.f;
  const int vq = L.valid ? __float2int_rn(q * p * kFixScale) : 0;   // pi in 2^-24 fixed point
  // inclusive scan of vq within the group (exact integer sums)
  int sc = vq;
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
  long long wl = 0, tpc = 0;
  if (L.valid) {
    const short4 e = __ldg(&P.sxy[L.sub]);
    const int x0 = e.x, y0 = e.y, x1 = e.z, y1 = e.w;
    const long long s = (y1 > y0) ? 1 : -1;
    const long long a = Av, bb = Bv, hs = S2 - S1, vs = Se - S2, v = vq;
    const int mid = (int)(L.pw >> 16);
    switch (L.shape) {
      case kStraightH: add_cell(P, x0, y0, v, 0, 0); add_cell(P, x1, y0, -v, 0, 0); tpc = 0; break;
      case kStraightV: add_cell(P, x0, y0, 0, v, 0); add_cell(P, x0, y1, 0, -v, 0); tpc = 0; break;
      case kHV:
        add_cell(P, x0, y0, a + hs, s * (bb + vs), 0);
        add_cell(P, x1, y0, -a, s * a, a);
        tpc = 1; break;
      case kVH:
        add_cell(P, x0, y1, bb, -s * bb, bb);
        add_cell(P, x1, y1, -(bb + hs), -s * (a + vs), 0);
        tpc = 1; break;
      case kZHVH:
        add_cell(P, mid, y0, -v, s * v, v);
        add_cell(P, mid, y1, v, -s * v, v);
        tpc = 2; break;
      default:  // kZVHV
        add_cell(P, x0, mid, v, -s * v, v);
        add_cell(P, x1, mid, -v, s * v, v);
        tpc = 2; break;
    }
    wl = (long long)vq * ((x1 - x0) + abs(y1 - y0));
    tpc *= vq;
  }
  // E[WL], E[TP] in fixed point: warp reduce, one atomic per warp
  wl = seg_reduce(wl, L.lane, 31, Sum());
  tpc = seg_reduce(tpc, L.lane, 31, Sum());
  if (L.lane == 0) { red64(P.scal, wl); red64(P.scal + 1, tpc); }
}

// ------------------------------------------------------------------------------------------
// KG: one CTA per line (Y H-rows, then X V-columns).  Scan of the difference array gives the
// wire demand W; d = (W + beta (VD_a + VD_b)) 2^-24 (Eq. (10), reading Q3); overflow cost
// f(cap - d) (Eq. (9)); G = dcost/dd = -a3 f'(cap - d); S = exclusive prefix of G (fp64).
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
  long long* diff = isH ? P.dH + (size_t)ln * P.X : P.dVT + (size_t)ln * P.Y;
  const float* cap = isH ? P.capH + (size_t)ln * P.X : P.capVT + (size_t)ln * P.Y;
  double* S = isH ? P.SH + (size_t)ln * P.X : P.SVT + (size_t)ln * P.Y;
  float* dout = isH ? P.dOutH + (size_t)ln * P.X : P.dOutVT + (size_t)ln * P.Y;
  // VD at position pos of this line
  const size_t vd_base = isH ? (size_t)ln * P.X : (size_t)ln;
  const size_t vd_step = isH ? 1 : (size_t)P.X;
  const double beta = A.beta;
  long long carryW = 0;
  double carryS = 0.0, of = 0.0;
  for (int c0 = 0; c0 < n; c0 += kGThreads * kGItems) {
    const int base = c0 + threadIdx.x * kGItems;
    long long v[kGItems];
#pragma unroll
    for (int i = 0; i < kGItems; ++i) v[i] = (base + i < n) ? diff[base + i] : 0;
    long long run = 0;
#pragma unroll
    for (int i = 0; i < kGItems; ++i) { run += v[i]; v[i] = run; }   // local inclusive
    long long totW;
    const long long offW = block_exclusive_scan(run, shl, &totW);
    double g[kGItems];
    double grun = 0.0;
#pragma unroll
    for (int i = 0; i < kGItems; ++i) {
      const int pos = base + i;
      double G = 0.0;
      if (pos < n - 1) {
        const long long W = carryW + offW + v[i];
        const long long vda = P.VD[vd_base + (size_t)pos * vd_step];
        const long long vdb = P.VD[vd_base + (size_t)(pos + 1) * vd_step];
        const double d = (double)W * kFixInv + beta * ((double)(vda + vdb) * kFixInv);
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
      const int pos = base + i;
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
  }
}

// ------------------------------------------------------------------------------------------
// KB: reverse + Adam.  c_i = a1 WL_i + a2 sqrt(L) TP_i + sum_{e in i} G_e
//                          + beta sum_{v in TP(i)} sum_{e incident to v} G_e
// with sum over a segment = S[hi] - S[lo] (O(1) per segment).  dp = q c; dw = (p/t)(dp - sum p dp);
// dq_j += p_i c_i (fixed point, per tree); Adam (torch semantics) on w_i.
// ------------------------------------------------------------------------------------------
struct SGrid {
  const double* SH;
  const double* SVT;
  int X, Y;
  __device__ __forceinline__ double h(int x, int y) const { return __ldg(&SH[(size_t)y * X + x]); }
  __device__ __forceinline__ double v(int x, int y) const { return __ldg(&SVT[(size_t)x * Y + y]); }
  // sum of G over the existing edges incident to G-cell (x,y)
  __device__ __forceinline__ double tp(int x, int y) const {
    return h(min(x + 1, X - 1), y) - h(max(x - 1, 0), y) + v(x, min(y + 1, Y - 1)) - v(x, max(y - 1, 0));
  }
};

__device__ __forceinline__ void adam_update(float& w, float& m, float& v, float g, const StepArgs& A) {
  m = fmaf(0.1f, g - m, m);                         // m.lerp_(g, 1 - beta1)
  v = fmaf(0.999f, v, 0.001f * g * g);              // v * beta2 + (1 - beta2) g^2
  const float denom = sqrtf(v) * A.inv_sqrt_bc2 + 1e-8f;
  w -= A.lr_over_bc1 * (m / denom);
}

__global__ void __launch_bounds__(256) kb_kernel(KParams P, StepArgs A) {
  const int b = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (b >= P.nb) return;
  Lane L;
  lane_setup(P, b, L);
  const size_t slot = (size_t)b * 32 + L.lane;
  float w = P.wp[slot];
  const float p = group_softmax(P, A, L, w);
  const float q = L.valid ? __ldg(&P.q[L.tree]) : 0.f;
  double c = 0.0;
  if (L.valid) {
    const SGrid S{P.SH, P.SVT, P.X, P.Y};
    const short4 e = __ldg(&P.sxy[L.sub]);
    const int x0 = e.x, y0 = e.y, x1 = e.z, y1 = e.w;
    const double s = (y1 > y0) ? 1.0 : -1.0;
    const int mid = (int)(L.pw >> 16);
    const double beta = A.beta;
    int ntp = 0;
    switch (L.shape) {
      case kStraightH: c = S.h(x1, y0) - S.h(x0, y0); break;
      case kStraightV: c = S.v(x0, y1) - S.v(x0, y0); break;
      case kHV:
        c = (S.h(x1, y0) - S.h(x0, y0)) + s * (S.v(x1, y1) - S.v(x1, y0)) + beta * S.tp(x1, y0);
        ntp = 1; break;
      case kVH:
        c = s * (S.v(x0, y1) - S.v(x0, y0)) + (S.h(x1, y1) - S.h(x0, y1)) + beta * S.tp(x0, y1);
        ntp = 1; break;
      case kZHVH:
        c = (S.h(mid, y0) - S.h(x0, y0)) + s * (S.v(mid, y1) - S.v(mid, y0)) + (S.h(x1, y1) - S.h(mid, y1)) +
            beta * (S.tp(mid, y0) + S.tp(mid, y1));
        ntp = 2; break;
      default:
        c = s * (S.v(x0, mid) - S.v(x0, y0)) + (S.h(x1, mid) - S.h(x0, mid)) + s * (S.v(x1, y1) - S.v(x1, mid)) +
            beta * (S.tp(x0, mid) + S.tp(x1, mid));
        ntp = 2; break;
    }
    c += (double)A.a_wl * (double)((x1 - x0) + abs(y1 - y0)) + (double)A.a_via * (double)A.sqrt_l * ntp;
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
  if (L.valid && ((th >> L.lane) & 1u)) red64(P.dq + L.tree, __double2ll_rn(pc * (double)kFixScale));
  if (L.valid) {
    float m = P.mp[slot], v = P.vp[slot];
    adam_update(w, m, v, (float)dw, A);
    P.wp[slot] = w;
    P.mp[slot] = m;
    P.vp[slot] = v;
  }
}

// ------------------------------------------------------------------------------------------
// KT: du_j = (q_j/t)(dq_j - sum_l q_l dq_l) over the net's trees; Adam on the tree logits.
// ------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) kt_kernel(KParams P, StepArgs A) {
  const int n = blockIdx.x * blockDim.x + threadIdx.x;
  if (n >= P.n_nets_l) return;
  const int a = P.net_tree_off[n], b = P.net_tree_off[n + 1];
  double sq = 0.0, sw = 0.0;
  for (int j = a; j < b; ++j) { sq += (double)P.q[j] * ((double)P.dq[j] * kFixInv); sw += (double)P.q[j]; }
  sq /= sw;   // weighted mean of dq (see the path-level softmax backward in kb_kernel)
  for (int j = a; j < b; ++j) {
    const double dqj = (double)P.dq[j] * kFixInv;
    P.dq[j] = 0;
    const double du = (b - a == 1) ? 0.0 : (double)P.q[j] * (double)A.inv_t * (dqj - sq);
    float w = P.wt[j], m = P.mt[j], v = P.vt[j];
    adam_update(w, m, v, (float)du, A);
    P.wt[j] = w; P.mt[j] = m; P.vt[j] = v;
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

void launch_kq(const KParams& p, const StepArgs& a, cudaStream_t s) {
  if (p.n_nets_l > 0) kq_kernel<<<cdiv(p.n_nets_l, 256), 256, 0, s>>>(p, a);
}
void launch_kf(const KParams& p, const StepArgs& a, cudaStream_t s) {
  if (p.nb > 0) kf_kernel<<<cdiv(p.nb, 8), 256, 0, s>>>(p, a);
}
void launch_kg(const KParams& p, const StepArgs& a, cudaStream_t s) {
  kg_kernel<<<p.X + p.Y, kGThreads, 0, s>>>(p, a);
  kg_finalize_kernel<<<1, 256, 0, s>>>(p, a);
}
void launch_kb(const KParams& p, const StepArgs& a, cudaStream_t s) {
  if (p.nb > 0) kb_kernel<<<cdiv(p.nb, 8), 256, 0, s>>>(p, a);
}
void launch_kt(const KParams& p, const StepArgs& a, cudaStream_t s) {
  if (p.n_nets_l > 0) kt_kernel<<<cdiv(p.n_nets_l, 256), 256, 0, s>>>(p, a);
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
