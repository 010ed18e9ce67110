// dgr_api.cu — libdgr's C ABI (include/dgr.h): validation, net sharding, device encoding,
// workspace layout, the iteration driver and the NCCL demand exchange.
//
// The data-parallel unit is the net (§3.2: nets couple only through the demand d of
// Eq. (10)).  Rank r keeps a contiguous, work-balanced range of nets; per iteration
// the ranks exchange one int64 buffer [dH | dV^T | E[WL], E[TP]] with ncclAllReduce —
// fixed point makes the sum exact, so every rank then runs the (replicated) grid pass on
// identical data and the result does not depend on the number of ranks.
#include <cuda_runtime.h>
#include <nccl.h>
#include <cuda.h>
#include <cudaTypedefs.h>
#include <map>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "dgr.h"
#include "dgr_internal.h"

using namespace dgr;

namespace {

thread_local std::string g_err;

int fail(int code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}

#define CUDA_TRY(x)                                                                          \
  do {                                                                                       \
    cudaError_t e_ = (x);                                                                    \
    if (e_ != cudaSuccess) return fail(DGR_ECUDA, "%s: %s", #x, cudaGetErrorString(e_));      \
  } while (0)
#define NCCL_TRY(x)                                                                          \
  do {                                                                                       \
    ncclResult_t r_ = (x);                                                                   \
    if (r_ != ncclSuccess) return fail(DGR_ENCCL, "%s: %s", #x, ncclGetErrorString(r_));      \
  } while (0)

// ---------------------------------------------------------------------------------------
// validation + sharding
// ---------------------------------------------------------------------------------------
int check_offsets(const int64_t* off, int64_t n, int64_t total, const char* name, bool nonempty) {
  if (!off) return fail(DGR_EINVAL, "%s is NULL", name);
  if (off[0] != 0) return fail(DGR_EINVAL, "%s[0] != 0", name);
  int64_t bad = n;   // first offending group (parallel scan, reported in index order)
#pragma omp parallel for schedule(static) reduction(min : bad)
  for (int64_t i = 0; i < n; ++i)
    if (off[i + 1] < off[i] || (nonempty && off[i + 1] == off[i])) bad = std::min(bad, i);
  if (bad < n) {
    if (off[bad + 1] < off[bad]) return fail(DGR_EINVAL, "%s not monotone at %lld", name, (long long)bad);
    return fail(DGR_EINVAL, "%s: empty group %lld", name, (long long)bad);
  }
  if (off[n] != total) return fail(DGR_EINVAL, "%s[n] = %lld != %lld", name, (long long)off[n], (long long)total);
  return DGR_OK;
}

int validate_structure(const dgr_forest_desc* d) {
  if (!d) return fail(DGR_EINVAL, "desc is NULL");
  if (d->X < 2 || d->Y < 2 || d->X > 32767 || d->Y > 32767) return fail(DGR_EINVAL, "grid must be 2..32767 per side");
  if (d->n_nets < 0 || d->n_trees < 0 || d->n_subnets < 0 || d->n_paths < 0 || d->n_segs < 0 || d->n_tps < 0)
    return fail(DGR_EINVAL, "negative count");
  if (d->n_paths >= (1ll << 31) || d->n_subnets >= (1ll << 31) || d->n_trees >= (1ll << 31))
    return fail(DGR_EINVAL, "more than 2^31 candidates");
  int rc;
  if ((rc = check_offsets(d->net_tree_off, d->n_nets, d->n_trees, "net_tree_off", true))) return rc;
  if ((rc = check_offsets(d->tree_sub_off, d->n_trees, d->n_subnets, "tree_sub_off", true))) return rc;
  if ((rc = check_offsets(d->sub_path_off, d->n_subnets, d->n_paths, "sub_path_off", true))) return rc;
  if ((rc = check_offsets(d->path_seg_off, d->n_paths, d->n_segs, "path_seg_off", true))) return rc;
  if ((rc = check_offsets(d->path_tp_off, d->n_paths, d->n_tps, "path_tp_off", false))) return rc;
  int64_t big = d->n_subnets;
#pragma omp parallel for schedule(static) reduction(min : big)
  for (int64_t s = 0; s < d->n_subnets; ++s)
    if (d->sub_path_off[s + 1] - d->sub_path_off[s] > kGenMaxGroup) big = std::min(big, s);
  if (big < d->n_subnets)
    return fail(DGR_EINVAL, "sub-net %lld has %lld > %d candidates", (long long)big,
                (long long)(d->sub_path_off[big + 1] - d->sub_path_off[big]), kGenMaxGroup);
  if ((d->n_segs && !d->seg) || (d->n_tps && !d->tp_xy) || (d->n_subnets && !d->sub_xy) || !d->cap_h ||
      !d->cap_v || (d->n_trees && !d->w_tree0) || (d->n_paths && !d->w_path0))
    return fail(DGR_EINVAL, "NULL array");
  return DGR_OK;
}

int partition(const dgr_forest_desc* d, int world, std::vector<int64_t>& out) {
  if (world < 1) return fail(DGR_EINVAL, "world < 1");
  out.assign(world + 1, 0);
  // work of a net = its paths + its segments (the per-candidate streams of KF / KB); the work of
  // nets [0, n) telescopes to first_path(n) + first_seg(first_path(n)), so cut points are binary
  // searches on that monotone function
  auto pref = [&](int64_t n) {
    const int64_t p = d->sub_path_off[d->tree_sub_off[d->net_tree_off[n]]];
    return p + d->path_seg_off[p];
  };
  const int64_t total = pref(d->n_nets);
  for (int r = 1; r < world; ++r) {
    const int64_t target = (int64_t)std::ceil((double)total * r / world);
    int64_t lo = out[r - 1], hi = d->n_nets;   // first n in [lo, n_nets] with pref(n) >= target
    while (lo < hi) {
      const int64_t mid = lo + (hi - lo) / 2;
      if (pref(mid) < target) lo = mid + 1; else hi = mid;
    }
    out[r] = lo;
  }
  out[world] = d->n_nets;
  return DGR_OK;
}

// ---------------------------------------------------------------------------------------
// pattern recognition: each explicit path must be a straight / L / Z pattern of its sub-net
// ---------------------------------------------------------------------------------------
struct Seg4 { int a, b, c, d; };
inline bool seg_eq(const Seg4& x, const Seg4& y) { return x.a == y.a && x.b == y.b && x.c == y.c && x.d == y.d; }

// Which pattern of sub-net (x0,y0)-(x1,y1) (canonical: x0 <= x1) path i is, and its x_m / y_m;
// *outside: a Z pattern whose x_m / y_m lies outside the sub-net's span (a C-shape detour, Q14b).
// The path's segments and turning points may come in any order: each expected one must be
// present and the counts must agree (the expected ones of a pattern are distinct, so a duplicate
// in the path leaves one uncovered).  The turning points fix the pattern; the segments confirm it.
bool classify(const dgr_forest_desc* d, int64_t i, int x0, int y0, int x1, int y1, uint32_t* shape, int* mid,
              bool* outside) {
  *outside = false;
  const int64_t g0 = d->path_seg_off[i], g1 = d->path_seg_off[i + 1];
  const int64_t t0 = d->path_tp_off[i], t1 = d->path_tp_off[i + 1];
  const int ns = (int)(g1 - g0), nt = (int)(t1 - t0);
  if (ns < 1 || ns > 3 || nt != ns - 1) return false;
  Seg4 segs[3];
  for (int g = 0; g < ns; ++g) {
    const int32_t* sg = d->seg + 4 * (g0 + g);
    segs[g] = {sg[0], sg[1], sg[2], sg[3]};
  }
  auto has = [&](const Seg4& e) {
    for (int q = 0; q < ns; ++q) if (seg_eq(segs[q], e)) return true;
    return false;
  };
  const int ylo = std::min(y0, y1), yhi = std::max(y0, y1);
  const int32_t* tp = d->tp_xy + 2 * t0;
  if (y0 == y1) {
    if (ns != 1 || !has({0, y0, x0, x1})) return false;
    *shape = kStraightH; *mid = 0; return true;
  }
  if (x0 == x1) {
    if (ns != 1 || !has({1, x0, ylo, yhi})) return false;
    *shape = kStraightV; *mid = 0; return true;
  }
  if (ns == 2) {
    if (tp[0] == x1 && tp[1] == y0 && has({0, y0, x0, x1}) && has({1, x1, ylo, yhi})) { *shape = kHV; *mid = 0; return true; }
    if (tp[0] == x0 && tp[1] == y1 && has({1, x0, ylo, yhi}) && has({0, y1, x0, x1})) { *shape = kVH; *mid = 0; return true; }
    return false;
  }
  if (ns != 3) return false;
  const int ax = tp[0], ay = tp[1], bx = tp[2], by = tp[3];
  if (ax == bx && ((ay == y0 && by == y1) || (ay == y1 && by == y0))) {   // Z-HVH (or C-HVH) at x_m = ax
    const int xm = ax;
    if (xm == x0 || xm == x1) return false;
    if (xm < 0 || xm >= d->X) return false;   // a C-shape detour must stay inside the grid
    if (!has({0, y0, std::min(x0, xm), std::max(x0, xm)}) || !has({1, xm, ylo, yhi}) ||
        !has({0, y1, std::min(xm, x1), std::max(xm, x1)}))
      return false;
    *shape = kZHVH; *mid = xm; *outside = xm < x0 || xm > x1; return true;
  }
  if (ay == by && ((ax == x0 && bx == x1) || (ax == x1 && bx == x0))) {   // Z-VHV (or C-VHV) at y_m = ay
    const int ym = ay;
    if (ym == y0 || ym == y1) return false;
    if (ym < 0 || ym >= d->Y) return false;   // a C-shape detour must stay inside the grid
    *outside = ym < ylo || ym > yhi;
    if (!has({1, x0, std::min(y0, ym), std::max(y0, ym)}) || !has({0, ym, x0, x1}) ||
        !has({1, x1, std::min(ym, y1), std::max(ym, y1)}))
      return false;
    *shape = kZVHV; *mid = ym; return true;
  }
  return false;
}

// A candidate outside the Z(o, m) patterns (row f4', reading Q14c) runs on the general path from
// its explicit segments and turning points: each segment must be a non-empty edge range of a grid
// line, each turning point a grid cell on one of the path's segments.
bool valid_path(const dgr_forest_desc* d, int64_t i) {
  const int64_t g0 = d->path_seg_off[i], g1 = d->path_seg_off[i + 1];
  for (int64_t g = g0; g < g1; ++g) {
    const int32_t* s = d->seg + 4 * g;
    const int n = s[0] == 0 ? d->X : d->Y, m = s[0] == 0 ? d->Y : d->X;   // line length, lines
    if ((s[0] != 0 && s[0] != 1) || s[1] < 0 || s[1] >= m || s[2] < 0 || s[2] >= s[3] || s[3] > n - 1) return false;
  }
  for (int64_t t = d->path_tp_off[i]; t < d->path_tp_off[i + 1]; ++t) {
    const int x = d->tp_xy[2 * t], y = d->tp_xy[2 * t + 1];
    if (x < 0 || x >= d->X || y < 0 || y >= d->Y) return false;
    bool on = false;
    for (int64_t g = g0; g < g1 && !on; ++g) {
      const int32_t* s = d->seg + 4 * g;
      on = s[0] == 0 ? (s[1] == y && s[2] <= x && x <= s[3]) : (s[1] == x && s[2] <= y && y <= s[3]);
    }
    if (!on) return false;
  }
  return true;
}

// ---------------------------------------------------------------------------------------
// the rank's encoded shard
// ---------------------------------------------------------------------------------------
// Uninitialised array of a trivially copyable type (the planner writes every element in parallel;
// std::vector would zero ~100 MB on one thread first).
template <class T>
struct PodBuf {
  std::unique_ptr<T[]> p;
  size_t n = 0;
  void alloc(size_t count) { p.reset(count ? new T[count] : nullptr); n = count; }
  void clear() { p.reset(); n = 0; }
  T* data() { return p.get(); }
  const T* data() const { return p.get(); }
  size_t size() const { return n; }
  T& operator[](size_t i) { return p[i]; }
  const T& operator[](size_t i) const { return p[i]; }
};

// Process-wide pinned staging buffer for the workspace upload (grow-only, reused by every handle;
// the driver's pageable copies would stage through a small bounce buffer instead).  Callers hold
// the lock from staging until their copies have completed.
struct PinnedPool {
  std::mutex m;
  char* p = nullptr;
  size_t n = 0;
  char* get(size_t bytes) {   // with m held
    if (bytes <= n) return p;
    if (p) cudaFreeHost(p);
    p = nullptr;
    n = 0;
    if (cudaHostAlloc(reinterpret_cast<void**>(&p), bytes, cudaHostAllocDefault) != cudaSuccess) { p = nullptr; return nullptr; }
    n = bytes;
    return p;
  }
};
PinnedPool g_pin;

// parallel copy into pinned staging memory
void par_copy(char* dst, const void* src, size_t bytes) {
  const char* s = static_cast<const char*>(src);
  constexpr size_t kChunk = 1 << 20;
  const int64_t nch = (int64_t)((bytes + kChunk - 1) / kChunk);
#pragma omp parallel for schedule(static)
  for (int64_t c = 0; c < nch; ++c) {
    const size_t o = (size_t)c * kChunk;
    memcpy(dst + o, s + o, std::min(kChunk, bytes - o));
  }
}

struct Plan {
  int64_t net_lo = 0, net_hi = 0, tree_lo = 0, tree_hi = 0, sub_lo = 0, sub_hi = 0, path_lo = 0, path_hi = 0;
  int64_t nid_base = 0;                 // global noise index of the rank's first noisy candidate
  int rank = 0, world = 1;
  int nb = 0;
  PodBuf<int4> binfo;
  PodBuf<uint32_t> pword;
  PodBuf<short4> sxy;                   // kernel order
  std::vector<int32_t> net_tree_off;   // over the nets in plan order: tree offsets in plan (tile) order
  std::vector<int64_t> perm;           // plan position -> local CSR net (spatial order, see make_plan 1c)
  std::vector<int32_t> tperm;          // plan-ordered local tree -> local CSR tree
  std::vector<int32_t> net_gtree;      // plan position -> local CSR index of the net's first tree
  std::vector<NoiseRun> runs;          // per tile (TileDesc run0 / nrun)
  std::vector<uint32_t> mnets;          // per tile: the trees of its nets with >= 2 trees, one per lane (tree_lane),
                                        // a net's trees never straddle a warp; padded to warps (TileDesc mn0 / nmn)
  PodBuf<int32_t> ksub_csr;             // kernel-order sub-net -> local CSR sub-net
  PodBuf<int64_t> sub_first_slot;       // local CSR sub-net -> slot of its first candidate
  PodBuf<int32_t> slot_path;            // slot -> local CSR path (-1: padding)
  PodBuf<uint32_t> ldesc;               // per bundle slot: lane descriptor (lane_desc)
  std::vector<TileDesc> tiles;          // pipelined tiles first (see make_plan)
  int64_t n_global_tiles = 0;
  int64_t n_pipe_tiles = 0;
  std::vector<std::pair<int, int>> tmap_shapes;   // (ww, wh) of each tensor-map pair (TileDesc::tmap)
  // general nets (row f4'): their candidates take virtual slots [nb * 32, nb * 32 + n_gpath)
  int64_t n_gpath = 0;
  std::vector<int2> gnet;
  std::vector<int4> gtree;
  std::vector<GSub> gsub;
  std::vector<int32_t> gp_seg_off, gp_tp_off;
  std::vector<short4> gseg;
  std::vector<short2> gtp;
};

// (cell, field) pairs of one candidate's demand events in the pipelined tile kernel (field 0 dH,
// 1 dV, 2 VD; see process_tile in dgr_kernels.cu): the Z(o, m) form's segment ends and turning
// points.  Returns their number (<= 8); zero-length segments emit nothing.
int lane_events(uint32_t pw, int x0, int y0, int x1, int y1, int ex[8], int ey[8], int ef[8]) {
  const int o = pw & 1, ntp = (pw >> 1) & 3, m = (int)(pw >> 16);
  const int p0 = o ? y0 : x0, p1 = o ? y1 : x1, q0 = o ? x0 : y0, q1 = o ? x1 : y1;
  int n = 0;
  auto ev = [&](int f, int p, int q) {   // (p, q) of orientation o -> (x, y)
    ex[n] = o ? q : p; ey[n] = o ? p : q; ef[n] = f; ++n;
  };
  if (m != p0) { ev(o, p0, q0); ev(o, m, q0); }
  if (p1 != m) { ev(o, m, q1); ev(o, p1, q1); }
  if (q1 != q0) { ev(1 - o, m, q0); ev(1 - o, m, q1); }
  if (ntp >= 1) ev(2, m, q0);
  if (ntp == 2) ev(2, m, q1);
  return n;
}

// A sub-net whose only candidate is one segment draws no noise and needs no softmax (Q7).
inline bool lone_straight(const dgr_forest_desc* d, int64_t s) {
  const int64_t p0 = d->sub_path_off[s];
  return d->sub_path_off[s + 1] - p0 == 1 && d->path_seg_off[p0 + 1] - d->path_seg_off[p0] == 1;
}

// Candidate order the forward's event collapse relies on (dgr.h): straight only if aligned, else
// HV, VH, Z-HVH..., Z-VHV..., then C-shapes (shapes[] carry kOutside)
inline bool canonical_group(const uint32_t* shapes, int n, bool aligned) {
  if (aligned) {
    for (int i = 0; i < n; ++i) if (shapes[i] != kStraightH && shapes[i] != kStraightV) return false;
    return true;
  }
  if (n < 2 || shapes[0] != kHV || shapes[1] != kVH) return false;
  int i = 2;
  while (i < n && shapes[i] == kZHVH) ++i;
  while (i < n && shapes[i] == kZVHV) ++i;
  while (i < n && (shapes[i] == (kZHVH | kOutside) || shapes[i] == (kZVHV | kOutside))) ++i;
  return i == n;
}

struct PhaseTimer {   // DGR_PLAN_TIMING=1: host planning phases to stderr (development aid)
  bool on = getenv("DGR_PLAN_TIMING") != nullptr;
  std::chrono::steady_clock::time_point t = std::chrono::steady_clock::now();
  void mark(const char* what) {
    if (!on) return;
    const auto n = std::chrono::steady_clock::now();
    fprintf(stderr, "[dgr plan] %-28s %8.2f ms\n", what, std::chrono::duration<double, std::milli>(n - t).count());
    t = n;
  }
};

int make_plan(const dgr_forest_desc* d, int rank, int world, Plan& pl) {
  PhaseTimer tm;
  pl.rank = rank;
  pl.world = world;
  int rc = validate_structure(d);
  tm.mark("validate");
  if (rc) return rc;
  std::vector<int64_t> part;
  if ((rc = partition(d, world, part))) return rc;
  tm.mark("partition");
  pl.net_lo = part[rank];
  pl.net_hi = part[rank + 1];
  pl.tree_lo = d->net_tree_off[pl.net_lo];
  pl.tree_hi = d->net_tree_off[pl.net_hi];
  pl.sub_lo = d->tree_sub_off[pl.tree_lo];
  pl.sub_hi = d->tree_sub_off[pl.tree_hi];
  pl.path_lo = d->sub_path_off[pl.sub_lo];
  pl.path_hi = d->sub_path_off[pl.sub_hi];
  const int64_t nn = pl.net_hi - pl.net_lo, ns = pl.sub_hi - pl.sub_lo;
  const int X = d->X, Y = d->Y;
  // noise indices: the candidates of earlier ranks' nets that draw noise
  {
    int64_t cnt = 0;
#pragma omp parallel for schedule(static) reduction(+ : cnt)
    for (int64_t s = 0; s < pl.sub_lo; ++s) cnt += lone_straight(d, s) ? 0 : d->sub_path_off[s + 1] - d->sub_path_off[s];
    pl.nid_base = cnt;
  }
  tm.mark("noise base");
  // 1. canonical sub-net endpoints + pattern words of every local candidate (parallel over
  //    sub-nets; the first failing sub-net, in index order, is reported)
  PodBuf<short4> sxy_csr, sub_ext;
  PodBuf<uint32_t> pw_path;
  PodBuf<char> single, gen;   // gen: the sub-net runs on the general path (row f4')
  sxy_csr.alloc(ns);
  sub_ext.alloc(ns);
  pw_path.alloc((size_t)(pl.path_hi - pl.path_lo));
  single.alloc(ns);
  gen.alloc(ns);
  int64_t bad_sub = ns;   // smallest failing local sub-net
#pragma omp parallel for schedule(dynamic, 4096) reduction(min : bad_sub)
  for (int64_t ls = 0; ls < ns; ++ls) {
    const int64_t s = pl.sub_lo + ls;
    const int32_t* e = d->sub_xy + 4 * s;
    int x0 = e[0], y0 = e[1], x1 = e[2], y1 = e[3];
    single[ls] = 0;
    gen[ls] = 0;
    if (x0 > x1 || (x0 == x1 && y0 > y1)) { std::swap(x0, x1); std::swap(y0, y1); }
    if (x0 < 0 || x1 >= X || std::min(y0, y1) < 0 || std::max(y0, y1) >= Y || (x0 == x1 && y0 == y1)) {
      bad_sub = std::min(bad_sub, ls);
      continue;
    }
    sxy_csr[ls] = make_short4((short)x0, (short)y0, (short)x1, (short)y1);
    const int64_t p0 = d->sub_path_off[s], p1 = d->sub_path_off[s + 1];
    uint32_t shapes[32];
    bool ok = p1 - p0 <= 32;
    int ex0 = x0, ex1 = x1, ey0 = std::min(y0, y1), ey1 = std::max(y0, y1);   // extent incl. detours
    for (int64_t i = p0; i < p1 && ok; ++i) {
      uint32_t shape;
      int mid;
      bool outside;
      if (!classify(d, i, x0, y0, x1, y1, &shape, &mid, &outside)) { ok = false; break; }
      shapes[i - p0] = shape | (outside ? kOutside : 0u);
      if (shape == kStraightH || shape == kHV) mid = x1;   // m = p1: the Z(o, m) form of path_cost
      if (shape == kStraightV || shape == kVH) mid = y1;
      pw_path[i - pl.path_lo] = shape | (outside ? kOutside : 0u) | ((uint32_t)mid << 16);
      if (outside && shape == kZHVH) { ex0 = std::min(ex0, mid); ex1 = std::max(ex1, mid); }
      if (outside && shape == kZVHV) { ey0 = std::min(ey0, mid); ey1 = std::max(ey1, mid); }
    }
    sub_ext[ls] = make_short4((short)ex0, (short)ey0, (short)ex1, (short)ey1);
    if (!ok || !canonical_group(shapes, (int)(p1 - p0), x0 == x1 || y0 == y1)) {
      // not all Z(o, m) patterns in the tile kernel's order, or more than 32: the general path
      // (explicit segments), provided every candidate is a well-formed rectilinear path
      for (int64_t i = p0; i < p1; ++i)
        if (!valid_path(d, i)) { bad_sub = std::min(bad_sub, ls); break; }
      gen[ls] = 1;
      single[ls] = (p1 - p0 == 1) && (d->path_seg_off[p0 + 1] - d->path_seg_off[p0] == 1);
      continue;
    }
    single[ls] = (p1 - p0 == 1) && (shapes[0] == kStraightH || shapes[0] == kStraightV);
  }
  if (bad_sub < ns) {
    const int64_t s = pl.sub_lo + bad_sub;
    const int32_t* e = d->sub_xy + 4 * s;
    int x0 = e[0], y0 = e[1], x1 = e[2], y1 = e[3];
    if (x0 > x1 || (x0 == x1 && y0 > y1)) { std::swap(x0, x1); std::swap(y0, y1); }
    if (x0 < 0 || x1 >= X || std::min(y0, y1) < 0 || std::max(y0, y1) >= Y)
      return fail(DGR_EINVAL, "sub-net %lld endpoints outside the grid", (long long)s);
    if (x0 == x1 && y0 == y1) return fail(DGR_EINVAL, "sub-net %lld has zero length", (long long)s);
    for (int64_t i = d->sub_path_off[s]; i < d->sub_path_off[s + 1]; ++i)
      if (!valid_path(d, i))
        return fail(DGR_EINVAL, "path %lld of sub-net %lld is malformed (a segment outside the grid or empty, or a turning point off the path)",
                    (long long)i, (long long)s);
    return fail(DGR_EINVAL, "sub-net %lld is malformed", (long long)s);
  }
  // a net with any general sub-net runs entirely on the general path (its trees' softmax and dq
  // stay in one warp)
  PodBuf<char> gen_net;
  gen_net.alloc(nn);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t ln = 0; ln < nn; ++ln) {
    const int64_t n = pl.net_lo + ln;
    const int64_t s0 = d->tree_sub_off[d->net_tree_off[n]], s1 = d->tree_sub_off[d->net_tree_off[n + 1]];
    bool g = false;
    for (int64_t sn = s0; sn < s1 && !g; ++sn) g = gen[sn - pl.sub_lo];
    gen_net[ln] = g;
    if (g) for (int64_t sn = s0; sn < s1; ++sn) gen[sn - pl.sub_lo] = 1;
  }
  int64_t n_gpath = 0;
#pragma omp parallel for schedule(static) reduction(+ : n_gpath)
  for (int64_t ls = 0; ls < ns; ++ls)
    if (gen[ls]) n_gpath += d->sub_path_off[pl.sub_lo + ls + 1] - d->sub_path_off[pl.sub_lo + ls];
  pl.n_gpath = n_gpath;
  tm.mark("classify");
  // local noise index of every sub-net's first candidate (-1 for lone straight paths)
  PodBuf<int64_t> nid_sub;
  nid_sub.alloc(ns);
  {
    // two-pass prefix over fixed chunks: noisy candidates per chunk, then the chunk offsets
    constexpr int64_t kChunk = 1 << 16;
    const int64_t nch = (ns + kChunk - 1) / kChunk;
    std::vector<int64_t> base(nch + 1, 0);
#pragma omp parallel for schedule(static)
    for (int64_t ch = 0; ch < nch; ++ch) {
      int64_t c = 0;
      for (int64_t ls = ch * kChunk; ls < std::min(ns, (ch + 1) * kChunk); ++ls)
        c += single[ls] ? 0 : d->sub_path_off[pl.sub_lo + ls + 1] - d->sub_path_off[pl.sub_lo + ls];
      base[ch + 1] = c;
    }
    for (int64_t ch = 0; ch < nch; ++ch) base[ch + 1] += base[ch];
#pragma omp parallel for schedule(static)
    for (int64_t ch = 0; ch < nch; ++ch) {
      int64_t next = base[ch];
      for (int64_t ls = ch * kChunk; ls < std::min(ns, (ch + 1) * kChunk); ++ls) {
        nid_sub[ls] = single[ls] ? -1 : next;
        next += single[ls] ? 0 : d->sub_path_off[pl.sub_lo + ls + 1] - d->sub_path_off[pl.sub_lo + ls];
      }
    }
  }
  // 2. tiles of whole nets: greedy in net order while the window (union of the nets' sub-net boxes
  //    plus a 1-cell halo) stays <= kWinMax cells, the group bundles <= kTargetBundles and all
  //    bundles <= kTileBundles, trees <= kPipeTrees, sub-nets <= kPipeSubs.  A net that alone
  //    exceeds the window forms a "global" tile.
  pl.tiles.clear();
  pl.binfo.clear();
  pl.pword.clear();
  // group bundles counted first-fit online (bin fills), singletons 32 to a bundle; the fill's packing
  // (pack_groups) never needs more bundles than this count
  struct Pack {
    int nbg = 0, nsing = 0;
    uint8_t fills[kMaxBundles];
    int total() const { return nbg + (nsing + 31) / 32; }
    void add(int g) {
      int k = 0;
      while (k < nbg && fills[k] + g > 32) ++k;
      if (k == nbg) {
        if (nbg == kMaxBundles) { ++nbg; return; }   // over the limit: the caller rejects the tile
        fills[nbg++] = 0;
      }
      fills[k] = (uint8_t)(fills[k] + g);
    }
  };
  struct Cur { bool open = false; int64_t net0 = 0; Pack pk; int ntree = 0, nsub = 0; int bx0 = 0, by0 = 0, bx1 = -1, by1 = -1; bool global = false; };
  // bounding box of each net's sub-nets plus a 1-cell halo (parallel over nets)
  PodBuf<int4> nbox;
  nbox.alloc(nn);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t ln = 0; ln < nn; ++ln) {
    const int64_t n = pl.net_lo + ln;
    int bx0 = X, by0 = Y, bx1 = -1, by1 = -1;
    const int64_t s0 = d->tree_sub_off[d->net_tree_off[n]], s1 = d->tree_sub_off[d->net_tree_off[n + 1]];
    for (int64_t s = s0; s < s1; ++s) {   // sub-net extents incl. C-shape detours
      const short4 e = sub_ext[s - pl.sub_lo];
      bx0 = std::min<int>(bx0, e.x); bx1 = std::max<int>(bx1, e.z);
      by0 = std::min<int>(by0, e.y); by1 = std::max<int>(by1, e.w);
    }
    nbox[ln] = make_int4(std::max(0, bx0 - 1), std::max(0, by0 - 1), std::min(X - 1, bx1 + 1), std::min(Y - 1, by1 + 1));
  }
  tm.mark("net boxes");
  // 1c. spatial order of the nets: tiles are runs of consecutive nets, so nets
  //     are taken in Morton order of their box centres, unless the caller's order is already
  //     spatially coherent (>= 80% of consecutive nets within 32 cells; forestgen emits Morton
  //     order) -- then that order.  Only the planning order changes: noise keys and every output
  //     stay in global (CSR) indices.
  std::vector<int64_t>& perm = pl.perm;
  perm.resize(nn);
  for (int64_t i = 0; i < nn; ++i) perm[i] = i;
  {
    int64_t near = 0;
#pragma omp parallel for schedule(static) reduction(+ : near)
    for (int64_t ln = 0; ln < nn - 1; ++ln) {
      const int4 a = nbox[ln], b = nbox[ln + 1];
      const int dx = std::abs((a.x + a.z) - (b.x + b.z)), dy = std::abs((a.y + a.w) - (b.y + b.w));   // 2 x centre distance
      near += std::max(dx, dy) <= 64;
    }
    const bool coherent = nn < 2 || near * 10 >= (nn - 1) * 8;
    if (!coherent || getenv("DGR_PLAN_SORT")) {
      auto spread = [](uint32_t v) {   // bit i -> bit 2i (16 bits)
        v &= 0xFFFF;
        v = (v | (v << 8)) & 0x00FF00FF; v = (v | (v << 4)) & 0x0F0F0F0F;
        v = (v | (v << 2)) & 0x33333333; v = (v | (v << 1)) & 0x55555555;
        return v;
      };
      std::vector<std::pair<uint32_t, int64_t>> key(nn);
#pragma omp parallel for schedule(static)
      for (int64_t ln = 0; ln < nn; ++ln) {
        const int4 b = nbox[ln];
        key[ln] = {spread((uint32_t)((b.x + b.z) >> 1)) | (spread((uint32_t)((b.y + b.w) >> 1)) << 1), ln};
      }
      std::sort(key.begin(), key.end());
      for (int64_t i = 0; i < nn; ++i) perm[i] = key[i].second;
    }
  }
  // trees and sub-nets renumbered in plan order (a tile's trees / sub-nets stay contiguous)
  std::vector<int32_t> ptree_off(nn + 1, 0), psub_off(nn + 1, 0);
  {   // counts, then a two-pass prefix over fixed chunks
#pragma omp parallel for schedule(static)
    for (int64_t pn = 0; pn < nn; ++pn) {
      const int64_t n = pl.net_lo + perm[pn];
      ptree_off[pn + 1] = (int32_t)(d->net_tree_off[n + 1] - d->net_tree_off[n]);
      psub_off[pn + 1] = (int32_t)(d->tree_sub_off[d->net_tree_off[n + 1]] - d->tree_sub_off[d->net_tree_off[n]]);
    }
    constexpr int64_t kChunk = 1 << 15;
    const int64_t nch = (nn + kChunk - 1) / kChunk;
    std::vector<int32_t> bt(nch + 1, 0), bs(nch + 1, 0);
#pragma omp parallel for schedule(static)
    for (int64_t ch = 0; ch < nch; ++ch) {
      int32_t a = 0, b = 0;
      for (int64_t pn = ch * kChunk + 1; pn <= std::min(nn, (ch + 1) * kChunk); ++pn) {
        a += ptree_off[pn]; ptree_off[pn] = a;
        b += psub_off[pn]; psub_off[pn] = b;
      }
      bt[ch + 1] = a; bs[ch + 1] = b;
    }
    for (int64_t ch = 0; ch < nch; ++ch) { bt[ch + 1] += bt[ch]; bs[ch + 1] += bs[ch]; }
#pragma omp parallel for schedule(static)
    for (int64_t ch = 1; ch < nch; ++ch)
      for (int64_t pn = ch * kChunk + 1; pn <= std::min(nn, (ch + 1) * kChunk); ++pn) {
        ptree_off[pn] += bt[ch];
        psub_off[pn] += bs[ch];
      }
  }
  pl.net_tree_off = ptree_off;
  pl.tperm.resize((size_t)(pl.tree_hi - pl.tree_lo));
  pl.net_gtree.resize(nn);
#pragma omp parallel for schedule(static)
  for (int64_t pn = 0; pn < nn; ++pn) {
    const int64_t n = pl.net_lo + perm[pn];
    pl.net_gtree[pn] = (int32_t)(d->net_tree_off[n] - pl.tree_lo);
    for (int64_t j = d->net_tree_off[n]; j < d->net_tree_off[n + 1]; ++j)
      pl.tperm[ptree_off[pn] + (j - d->net_tree_off[n])] = (int32_t)(j - pl.tree_lo);
  }
  tm.mark("spatial order");
  auto net_box = [&](int64_t n, int& bx0, int& by0, int& bx1, int& by1) {
    const int4 b = nbox[n - pl.net_lo];
    bx0 = b.x; by0 = b.y; bx1 = b.z; by1 = b.w;
  };
  auto pack_net = [&](int64_t n, Pack& pk) {   // bundle packing of one net's sub-nets
    const int64_t s0 = d->tree_sub_off[d->net_tree_off[n]], s1 = d->tree_sub_off[d->net_tree_off[n + 1]];
    for (int64_t s = s0; s < s1; ++s) {
      if (gen[s - pl.sub_lo]) continue;   // general path: virtual slots
      if (single[s - pl.sub_lo]) { ++pk.nsing; continue; }
      pk.add((int)(d->sub_path_off[s + 1] - d->sub_path_off[s]));
    }
  };
  // windows start on even cells and have even extents so their S rows / columns are 16-byte
  // aligned for the bulk (TMA) copies (the S arrays have an even pitch)
  auto aligned_area = [](int bx0, int by0, int bx1, int by1) -> int64_t {
    const int x0 = bx0 & ~1, y0 = by0 & ~1;
    const int w = (bx1 + 1 - x0 + 1) & ~1, h = (by1 + 1 - y0 + 1) & ~1;
    return std::max((int64_t)h * win_pitch(w), (int64_t)w * win_pitch(h));   // the padded fields (win_pitch)
  };
  // The greedy restarts at fixed chunk boundaries (independent of the thread count) so the chunks
  // run in parallel; each boundary costs at most one extra tile.
  constexpr int64_t kChunkNets = 1 << 15;
  const int64_t nchunk = std::max<int64_t>(1, (nn + kChunkNets - 1) / kChunkNets);
  // group bundles per tile: kTargetBundles, fewer for a forest too small to fill one wave of
  // resident tiles (148 SMs x 5 CTAs): there a tile's lifetime IS the kernel's time, and smaller
  // tiles cut it.  DGR_TILE_BUNDLES overrides (experiments).
  int tgt = kTargetBundles;
  {
    const int64_t est = (pl.path_hi - pl.path_lo + 31) / 32;   // ~ bundles of the rank's forest
    const int64_t slots = 148 * 5;
    if (est < (int64_t)kTargetBundles * slots) tgt = (int)std::max<int64_t>(4, (est + slots - 1) / slots);
    if (const char* e = getenv("DGR_TILE_BUNDLES")) tgt = std::min(kTargetBundles, std::max(1, atoi(e)));
  }
  std::vector<std::vector<int64_t>> cstarts(nchunk);
  std::vector<std::vector<char>> cglobs(nchunk);
  std::vector<int64_t> cbad(nchunk, -1);
  auto greedy = [&](const int tgt) {
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t ch = 0; ch < nchunk; ++ch) {
    cstarts[ch].clear();
    cglobs[ch].clear();
    cbad[ch] = -1;
    const int64_t pa = ch * kChunkNets, pb = std::min(nn, pa + kChunkNets);
    Cur cur;
    for (int64_t pn = pa; pn < pb; ++pn) {
      const int64_t n = pl.net_lo + perm[pn];
      if (gen_net[n - pl.net_lo]) {   // a general net: a "tile" of its own (global = 2, no bundles)
        cstarts[ch].push_back(pn);
        cglobs[ch].push_back(2);
        cur = Cur();
        continue;
      }
      int bx0, by0, bx1, by1;
      net_box(n, bx0, by0, bx1, by1);
      const bool big = aligned_area(bx0, by0, bx1, by1) > kWinMax;
      const int ntree = (int)(d->net_tree_off[n + 1] - d->net_tree_off[n]);
      const int nsub = (int)(d->tree_sub_off[d->net_tree_off[n + 1]] - d->tree_sub_off[d->net_tree_off[n]]);
      bool fits = cur.open && !cur.global && !big;
      Pack pk2 = cur.pk;
      if (fits) {
        const int ux0 = std::min(cur.bx0, bx0), uy0 = std::min(cur.by0, by0);
        const int ux1 = std::max(cur.bx1, bx1), uy1 = std::max(cur.by1, by1);
        pack_net(n, pk2);
        fits = aligned_area(ux0, uy0, ux1, uy1) <= kWinMax && pk2.nbg <= tgt && pk2.total() <= tgt + (kTileBundles - kTargetBundles) &&
               cur.ntree + ntree <= kPipeTrees && cur.nsub + nsub <= kPipeSubs;
        if (fits) { cur.bx0 = ux0; cur.by0 = uy0; cur.bx1 = ux1; cur.by1 = uy1; }
      } else if (cur.open && cur.global && big) {
        pack_net(n, pk2);
        fits = pk2.total() <= kMaxBundles && cur.ntree + ntree <= kTreeMax;
      }
      if (fits) {
        cur.pk = pk2; cur.ntree += ntree; cur.nsub += nsub;
        continue;
      }
      // close the open tile, open a new one at net n
      cstarts[ch].push_back(pn);
      cglobs[ch].push_back(big);
      cur = Cur();
      cur.open = true; cur.global = big; cur.net0 = pn; cur.ntree = ntree; cur.nsub = nsub;
      cur.bx0 = bx0; cur.by0 = by0; cur.bx1 = bx1; cur.by1 = by1;
      pack_net(n, cur.pk);
      if ((cur.pk.total() > kMaxBundles || ntree > kTreeMax) && cbad[ch] < 0) cbad[ch] = n;
    }
  }
  };
  greedy(tgt);
  // Between one and three waves of resident tiles the last wave runs part-empty: shrink the tiles
  // so the pipelined tiles fill whole waves (ispd18-sized forests: 1.45 waves of 32-bundle tiles ->
  // 24-bundle tiles, +3% same-box, profiles/r02_ab_tile_target_waves.jsonl)
  if (tgt == kTargetBundles && !getenv("DGR_TILE_BUNDLES")) {
    int64_t npipe = 0;
    for (int64_t ch = 0; ch < nchunk; ++ch)
      for (char g : cglobs[ch]) npipe += (g == 0);
    const double waves = (double)npipe / (148.0 * 5.0);
    if (waves > 1.0 && waves < 3.0) {
      const int t2 = std::max(16, (int)std::ceil(kTargetBundles * waves / std::ceil(waves)));
      if (t2 < tgt) greedy(t2);
    }
  }
  std::vector<int64_t> starts;
  std::vector<char> globs;
  for (int64_t ch = 0; ch < nchunk; ++ch) {
    if (cbad[ch] >= 0) {
      const int64_t n = cbad[ch];
      const int ntree = (int)(d->net_tree_off[n + 1] - d->net_tree_off[n]);
      if (ntree > kTreeMax) return fail(DGR_EINVAL, "net %lld has %d > %d trees", (long long)n, ntree, kTreeMax);
      Pack pk;
      pack_net(n, pk);
      return fail(DGR_EINVAL, "net %lld needs %d > %d bundles", (long long)n, pk.total(), kMaxBundles);
    }
    starts.insert(starts.end(), cstarts[ch].begin(), cstarts[ch].end());
    globs.insert(globs.end(), cglobs[ch].begin(), cglobs[ch].end());
  }
  starts.push_back(nn);   // plan positions
  tm.mark("tiles (greedy)");
  // Group bundles of a tile: its noisy sub-nets (groups of g <= 32 candidates, never split) packed
  // first-fit decreasing (ties in plan order), or first-fit in plan order when that needs fewer
  // bundles (so never more than the tile greedy's first-fit count).  Returns the bins as lists of indices into the tile's groups in plan order.
  // (no per-call allocations once warm: sizes bucketed 32..0 for the decreasing order, which keeps
  // plan order among equal sizes like a stable sort; the result is each group's bin, and the
  // members listed bin by bin in plan order)
  struct GroupPack {
    std::vector<int> bin_nf, bin_ff, fills, members, start, cursor;
    std::vector<int> bucket[33];
    int nbins = 0;
    void run(const std::vector<int>& gs) {
      const int n = (int)gs.size();
      fills.resize(n + 1);
      auto first_fit = [&](int g, int& nb) {
        int k = 0;
        while (k < nb && fills[k] + g > 32) ++k;
        if (k == nb) fills[nb++] = 0;
        fills[k] += g;
        return k;
      };
      bin_nf.resize(n); bin_ff.resize(n);
      int nnf = 0, nff = 0;
      for (int i = 0; i < n; ++i) bin_nf[i] = first_fit(gs[i], nnf);   // online, plan order (the greedy's count)
      for (auto& b : bucket) b.clear();
      for (int i = 0; i < n; ++i) bucket[std::min(gs[i], 32)].push_back(i);
      for (int g = 32; g >= 0; --g)
        for (int i : bucket[g]) bin_ff[i] = first_fit(gs[i], nff);
      const std::vector<int>& bin = nff <= nnf ? bin_ff : bin_nf;
      nbins = std::min(nff, nnf);
      start.assign(nbins + 1, 0);
      for (int i = 0; i < n; ++i) ++start[bin[i] + 1];
      for (int b = 0; b < nbins; ++b) start[b + 1] += start[b];
      cursor.assign(start.begin(), start.end() - 1);
      members.resize(n);
      for (int i = 0; i < n; ++i) members[cursor[bin[i]]++] = i;
    }
  };
  auto tile_groups = [&](int64_t pa, int64_t pb, std::vector<int>& gs) {   // group sizes of the tile's noisy sub-nets, plan order
    gs.clear();
    for (int64_t pn = pa; pn < pb; ++pn) {
      const int64_t n = pl.net_lo + perm[pn];
      const int64_t s0 = d->tree_sub_off[d->net_tree_off[n]], s1 = d->tree_sub_off[d->net_tree_off[n + 1]];
      for (int64_t sn = s0; sn < s1; ++sn)
        if (!gen[sn - pl.sub_lo] && !single[sn - pl.sub_lo]) gs.push_back((int)(d->sub_path_off[sn + 1] - d->sub_path_off[sn]));
    }
  };
  // 3. bundles, tile by tile: the tile's group bundles (packing restarts at each tile), then its
  //    singleton bundles; sub-nets renumbered in that order ("kernel order").  Count per tile,
  //    prefix, then fill the tiles in parallel (each owns a contiguous bundle and sub-net range).
  const int64_t ntile = (int64_t)starts.size() - 1;
  std::vector<int32_t> tb0(ntile + 1, 0), tbg(ntile, 0), tmn(ntile + 1, 0);
#pragma omp parallel
  {
  GroupPack gp;
  std::vector<int> gsz;
#pragma omp for schedule(dynamic, 64)
  for (int64_t t = 0; t < ntile; ++t) {
    Pack pk;
    int lanes = 0;   // tree lanes of the tile's multi-tree nets (a net's trees within one warp)
    for (int64_t pn = starts[t]; pn < starts[t + 1]; ++pn) {
      const int64_t n = pl.net_lo + perm[pn];
      pack_net(n, pk);
      const int nt = (int)(d->net_tree_off[n + 1] - d->net_tree_off[n]);
      if (nt > 1) {
        if ((lanes & 31) + nt > 32) lanes = (lanes + 31) & ~31;
        lanes += nt;
      }
    }
    tmn[t + 1] = (lanes + 31) & ~31;
    tile_groups(starts[t], starts[t + 1], gsz);
    gp.run(gsz);
    tbg[t] = (int32_t)gp.nbins;
    tb0[t + 1] = tbg[t] + (pk.nsing + 31) / 32;
  }
  }
  for (int64_t t = 0; t < ntile; ++t) { tb0[t + 1] += tb0[t]; tmn[t + 1] += tmn[t]; }
  pl.mnets.assign(tmn[ntile], 0);
  const size_t nslot = (size_t)tb0[ntile] * 32;
  // every element is written by the parallel fill below (padding slots included)
  pl.binfo.alloc(tb0[ntile]);
  pl.pword.alloc(nslot);
  pl.slot_path.alloc(nslot + (size_t)pl.n_gpath);   // bundle slots, then the general paths' virtual slots
  pl.ldesc.alloc(nslot);
  pl.sxy.alloc(ns);
  pl.ksub_csr.alloc(ns);
  pl.sub_first_slot.alloc(ns);
  pl.tiles.assign(ntile, TileDesc{});
  std::vector<std::vector<NoiseRun>> tile_runs(ntile);
  tm.mark("bundle counts + alloc");
#pragma omp parallel
  {
    std::vector<uint16_t> cnt;
    std::vector<int> stamp, cov;
    GroupPack gp;
    struct TT { int64_t j; int32_t pt; bool multi; };
    struct Grp { int64_t ls; int g, noff, toff; uint32_t mt; };
    std::vector<TT> tts;   // (per-thread buffers, reused across tiles)
    std::vector<Grp> grps;
    std::vector<int> gsz;
#pragma omp for schedule(dynamic, 16)
    for (int64_t t = 0; t < ntile; ++t) {
      TileDesc T{};
      T.net0 = (int32_t)starts[t];
      T.nnet = (int32_t)(starts[t + 1] - starts[t]);
      T.tree0 = ptree_off[starts[t]];
      T.ntree = ptree_off[starts[t + 1]] - T.tree0;
      // the tile's trees in plan order: CSR tree, plan-ordered local tree, net has >= 2 trees
      tts.clear();
      for (int64_t pn = starts[t]; pn < starts[t + 1]; ++pn) {
        const int64_t n = pl.net_lo + perm[pn];
        const int64_t a = d->net_tree_off[n], b = d->net_tree_off[n + 1];
        for (int64_t j = a; j < b; ++j) tts.push_back({j, (int32_t)(ptree_off[pn] + (j - a)), b - a > 1});
      }
      T.b0 = tb0[t];
      T.nb = tb0[t + 1] - tb0[t];
      T.mn0 = tmn[t];
      T.nmn = tmn[t + 1] - tmn[t];
      {
        int64_t k = T.mn0;
        for (int64_t pn = starts[t]; pn < starts[t + 1]; ++pn) {
          const int64_t n = pl.net_lo + perm[pn];
          const int nt = (int)(d->net_tree_off[n + 1] - d->net_tree_off[n]);
          if (nt < 2) continue;
          if (((k - T.mn0) & 31) + nt > 32)
            while ((k - T.mn0) & 31) pl.mnets[k++] = kNoTreeLane;
          for (int q = 0; q < nt; ++q)
            pl.mnets[k++] = tree_lane(ptree_off[pn] + q - T.tree0, (int)(pn - starts[t]), q == 0);
        }
        while (k < T.mn0 + T.nmn) pl.mnets[k++] = kNoTreeLane;
      }
      T.nbg = tbg[t];
      T.global = globs[t];
      int bx0 = X, by0 = Y, bx1 = -1, by1 = -1;
      for (int64_t pn = starts[t]; pn < starts[t + 1]; ++pn) {
        int a0, b0_, a1, b1_;
        net_box(pl.net_lo + perm[pn], a0, b0_, a1, b1_);
        bx0 = std::min(bx0, a0); by0 = std::min(by0, b0_); bx1 = std::max(bx1, a1); by1 = std::max(by1, b1_);
      }
      T.wx0 = bx0 & ~1; T.wy0 = by0 & ~1;
      T.ww = (bx1 + 1 - T.wx0 + 1) & ~1; T.wh = (by1 + 1 - T.wy0 + 1) & ~1;
      if (T.global) { T.wx0 = 0; T.wy0 = 0; T.ww = 0; T.wh = 0; }
      T.sub0 = psub_off[starts[t]];
      T.nsub = psub_off[starts[t + 1]] - T.sub0;
      for (int b = T.b0; b < T.b0 + T.nb; ++b) {
        pl.binfo[b] = make_int4(0, 0, 0, 0);
        for (int l = 0; l < 32; ++l) {
          pl.pword[(size_t)b * 32 + l] = kPad | kSubHead;
          pl.slot_path[(size_t)b * 32 + l] = -1;
          pl.ldesc[(size_t)b * 32 + l] = lane_desc(0, l, l, l);   // padding: a group of its own
        }
      }
      int ks = T.sub0;   // next kernel-order sub-net
      if (T.global == 2) {   // a general net: kernel order = CSR order; virtual slots assigned below
        for (const TT& tt : tts)
          for (int64_t sn = d->tree_sub_off[tt.j]; sn < d->tree_sub_off[tt.j + 1]; ++sn, ++ks) {
            pl.sxy[ks] = sxy_csr[sn - pl.sub_lo];
            pl.ksub_csr[ks] = (int32_t)(sn - pl.sub_lo);
          }
        pl.tiles[t] = T;
        continue;
      }
      // group bundles.  The tile's noisy sub-nets in plan order define the tile noise offsets, whose
      // global noise indices form runs (tile_noise fills gp by offset); the groups are then packed
      // (pack_groups), and each slot's lane descriptor carries its noise offset, group head and end
      // lane and its sub-net's index in the bundle (kernel order follows the bundles' slot order)
      grps.clear();
      gsz.clear();
      std::vector<NoiseRun> truns;
      int noff = 0;
      for (const TT& tt : tts) {
        for (int64_t sn = d->tree_sub_off[tt.j]; sn < d->tree_sub_off[tt.j + 1]; ++sn) {
          const int64_t ls = sn - pl.sub_lo;
          if (single[ls]) continue;
          const int g = (int)(d->sub_path_off[sn + 1] - d->sub_path_off[sn]);
          if (!truns.empty() && truns.back().nid + truns.back().len == (int32_t)nid_sub[ls]) truns.back().len += g;
          else truns.push_back({noff, g, (int32_t)nid_sub[ls], 0});
          grps.push_back({ls, g, noff, tt.pt - T.tree0, tt.multi ? kMultiTree : 0u});
          gsz.push_back(g);
          noff += g;
        }
      }
      gp.run(gsz);
      int b = T.b0 - 1, prev_tree = -1;
      for (int bn = 0; bn < gp.nbins; ++bn) {
        ++b;
        pl.binfo[b] = make_int4(0, ks, T.tree0, 0);
        int fill = 0, gi = 0;
        prev_tree = -1;
        for (int mi = gp.start[bn]; mi < gp.start[bn + 1]; ++mi) {
          const int idx = gp.members[mi];
          const Grp& G = grps[idx];
          const int64_t sn = pl.sub_lo + G.ls;
          const int64_t p0 = d->sub_path_off[sn], p1 = d->sub_path_off[sn + 1];
          pl.sxy[ks] = sxy_csr[G.ls];
          pl.ksub_csr[ks] = (int32_t)G.ls;
          pl.sub_first_slot[G.ls] = (int64_t)b * 32 + fill;
          for (int64_t i = p0; i < p1; ++i) {
            uint32_t pw = pw_path[i - pl.path_lo] | ((uint32_t)G.toff << kTreeShift) | G.mt;
            if (i == p0) {
              pw |= kSubHead;
              if (G.toff != prev_tree) pw |= kTreeHead;
            }
            const size_t slot = (size_t)b * 32 + fill + (i - p0);
            pl.pword[slot] = pw;
            pl.slot_path[slot] = (int32_t)(i - pl.path_lo);
            pl.ldesc[slot] = lane_desc(G.noff + (int)(i - p0), fill, fill + G.g - 1, gi);
          }
          prev_tree = G.toff;
          fill += G.g;
          pl.binfo[b].w += G.g;
          ++ks;
          ++gi;
        }
      }
      // singleton bundles: the lone straight sub-nets of multi-tree nets first, then those of
      // single-tree nets, so that most singleton bundles have no dq to accumulate (their reverse is
      // skipped)
      int lane = 32;
      b = T.b0 + T.nbg - 1;
      for (int pass = 0; pass < 2; ++pass)
      for (const TT& tt : tts) {
        const int64_t j = tt.j;
        const bool mj = tt.multi;
        if (mj != (pass == 0)) continue;
        const uint32_t mt = mj ? kMultiTree : 0u;
        const int toff = tt.pt - T.tree0;
        for (int64_t sn = d->tree_sub_off[j]; sn < d->tree_sub_off[j + 1]; ++sn) {
          const int64_t ls = sn - pl.sub_lo;
          if (!single[ls]) continue;
          if (lane == 32) {
            ++b;
            pl.binfo[b] = make_int4(0, ks, T.tree0, kSingleBundle);
            lane = 0;
            prev_tree = -1;
          }
          pl.sxy[ks] = sxy_csr[ls];
          pl.ksub_csr[ks] = (int32_t)ls;
          const int64_t p0 = d->sub_path_off[sn];
          const size_t slot = (size_t)b * 32 + lane;
          pl.sub_first_slot[ls] = (int64_t)slot;
          pl.pword[slot] = pw_path[p0 - pl.path_lo] | ((uint32_t)toff << kTreeShift) | kSubHead | mt |
                           (toff != prev_tree ? kTreeHead : 0u);
          pl.ldesc[slot] = lane_desc(0, lane, lane, lane);
          pl.slot_path[slot] = (int32_t)(p0 - pl.path_lo);
          prev_tree = toff;
          ++lane;
          pl.binfo[b].w += 1;
          ++ks;
        }
      }
      // int32 shared-memory accumulation is exact while no window cell-field is touched by more
      // than kEventMax sub-nets: the events one sub-net puts on one cell-field sum to at most
      // sum_j |pi_j| <= 2^24 + 32 in magnitude.  Otherwise run the tile against global memory.
      // Fast sufficient test first: a sub-net's events all lie inside its box (detours included),
      // so if no window cell is covered by more than kEventMax sub-net boxes (2-D difference array
      // over the window), no cell-field can be touched by more than kEventMax sub-nets.
      bool safe = false;
      if (!T.global) {
        const int W1 = T.ww + 1;
        cov.assign((size_t)W1 * (T.wh + 1), 0);
        for (const TT& tt : tts)
        for (int64_t sn = d->tree_sub_off[tt.j]; sn < d->tree_sub_off[tt.j + 1]; ++sn) {
          const short4 b = sub_ext[sn - pl.sub_lo];
          const int bx0 = b.x - T.wx0, by0 = b.y - T.wy0, bx1 = b.z - T.wx0 + 1, by1 = b.w - T.wy0 + 1;
          cov[(size_t)by0 * W1 + bx0] += 1; cov[(size_t)by0 * W1 + bx1] -= 1;
          cov[(size_t)by1 * W1 + bx0] -= 1; cov[(size_t)by1 * W1 + bx1] += 1;
        }
        int mx = 0;
        for (int y = 0; y < T.wh; ++y)
          for (int x = 0; x < T.ww; ++x) {
            int& c = cov[(size_t)y * W1 + x];
            c += (x > 0 ? cov[(size_t)y * W1 + x - 1] : 0) + (y > 0 ? cov[(size_t)(y - 1) * W1 + x] : 0) -
                 (x > 0 && y > 0 ? cov[(size_t)(y - 1) * W1 + x - 1] : 0);
            mx = std::max(mx, c);
          }
        safe = mx <= kEventMax;
      }
      if (!T.global && !safe) {
        cnt.assign((size_t)3 * T.ww * T.wh, 0);
        stamp.assign((size_t)3 * T.ww * T.wh, -1);   // last sub-net counted at a cell-field
        bool ok = true;
        int id = -1;
        for (const TT& tt : tts)
        for (int64_t sn = d->tree_sub_off[tt.j]; sn < d->tree_sub_off[tt.j + 1] && ok; ++sn) {
          const short4 e = sxy_csr[sn - pl.sub_lo];
          ++id;
          for (int64_t i = d->sub_path_off[sn]; i < d->sub_path_off[sn + 1] && ok; ++i) {
            const uint32_t pw = pw_path[i - pl.path_lo];
            int ex[8], ey[8], ef[8];
            const int ne = lane_events(pw, e.x, e.y, e.z, e.w, ex, ey, ef);
            for (int q = 0; q < ne; ++q) {
              // the event windows of the H / VD fields are row-major, the V field's column-major;
              // any fixed cell index works for counting
              const size_t c = (size_t)ef[q] * T.ww * T.wh + (size_t)(ey[q] - T.wy0) * T.ww + (ex[q] - T.wx0);
              if (stamp[c] != id) {
                stamp[c] = id;
                if (++cnt[c] > kEventMax) ok = false;
              }
            }
          }
        }
        if (!ok) { T.global = 1; T.wx0 = T.wy0 = T.ww = T.wh = 0; }
      }
      tile_runs[t] = std::move(truns);
      pl.tiles[t] = T;
    }
  }
  // the tiles' noise runs.  A tile with one run (the caller's order kept) draws its quads in
  // parallel from TileDesc alone; a tile with several (re-ordered nets: about one per net) gets its
  // runs cut at global noise indices that are multiples of 16, so each piece spans at most 4 Philox
  // quads and one thread draws it (no search for a quad's run)
  pl.runs.clear();
  for (int64_t t = 0; t < ntile; ++t) {
    TileDesc& T = pl.tiles[t];
    const auto& tr = tile_runs[t];
    T.run0 = (int32_t)pl.runs.size();
    T.nid0 = tr.empty() ? 0 : tr[0].nid;
    T.nnoisy = 0;
    for (const NoiseRun& r : tr) T.nnoisy += r.len;
    if (tr.size() <= 1) {
      T.nrun = (int32_t)tr.size();
      const int64_t g0 = pl.nid_base + T.nid0;
      T.nquad = tr.empty() ? 0 : (int32_t)(((g0 + T.nnoisy - 1) >> 2) - (g0 >> 2) + 1);
      for (const NoiseRun& r : tr) pl.runs.push_back(r);
      continue;
    }
    for (const NoiseRun& r : tr) {
      int off = r.off, nid = r.nid, len = r.len;
      while (len > 0) {
        const int64_t g = pl.nid_base + nid;
        const int piece = (int)std::min<int64_t>(len, 16 - (g & 15));
        pl.runs.push_back({off, piece, nid, 0});
        off += piece; nid += piece; len -= piece;
      }
    }
    T.nrun = (int32_t)(pl.runs.size() - T.run0);
    T.nquad = 0;
  }
  tm.mark("bundles + event check");
  pl.nb = (int)pl.binfo.size();
  // general nets (row f4'): out of the tile list into their own arrays, candidates on virtual slots
  {
    int64_t vslot = (int64_t)pl.nb * 32, gp = 0;
    pl.gp_seg_off.assign(1, 0);
    pl.gp_tp_off.assign(1, 0);
    for (const TileDesc& T : pl.tiles) {
      if (T.global != 2) continue;
      const int64_t n = pl.net_lo + perm[T.net0];
      const int64_t j0 = d->net_tree_off[n], j1 = d->net_tree_off[n + 1];
      pl.gnet.push_back(make_int2((int)pl.gtree.size(), (int)(j1 - j0)));
      int ks = T.sub0;
      for (int64_t j = j0; j < j1; ++j) {
        // {plan-ordered local tree, first gsub, sub-nets, local CSR tree (the tree's noise key)}
        pl.gtree.push_back(make_int4(T.tree0 + (int)(j - j0), (int)pl.gsub.size(),
                                     (int)(d->tree_sub_off[j + 1] - d->tree_sub_off[j]), (int)(j - pl.tree_lo)));
        for (int64_t sn = d->tree_sub_off[j]; sn < d->tree_sub_off[j + 1]; ++sn, ++ks) {
          const int64_t ls = sn - pl.sub_lo, p0 = d->sub_path_off[sn], p1 = d->sub_path_off[sn + 1];
          GSub g{};
          g.slot = (int32_t)vslot; g.n = (int32_t)(p1 - p0); g.nid = single[ls] ? -1 : (int32_t)nid_sub[ls];
          g.ksub = ks; g.tree = T.tree0 + (int32_t)(j - j0); g.gp = (int32_t)gp;
          pl.gsub.push_back(g);
          pl.sub_first_slot[ls] = vslot;
          for (int64_t i = p0; i < p1; ++i, ++vslot, ++gp) {
            pl.slot_path[vslot] = (int32_t)(i - pl.path_lo);
            for (int64_t q = d->path_seg_off[i]; q < d->path_seg_off[i + 1]; ++q) {
              const int32_t* sg = d->seg + 4 * q;
              pl.gseg.push_back(make_short4((short)sg[0], (short)sg[1], (short)sg[2], (short)sg[3]));
            }
            for (int64_t q = d->path_tp_off[i]; q < d->path_tp_off[i + 1]; ++q)
              pl.gtp.push_back(make_short2((short)d->tp_xy[2 * q], (short)d->tp_xy[2 * q + 1]));
            pl.gp_seg_off.push_back((int32_t)pl.gseg.size());
            pl.gp_tp_off.push_back((int32_t)pl.gtp.size());
          }
        }
      }
    }
    pl.tiles.erase(std::remove_if(pl.tiles.begin(), pl.tiles.end(), [](const TileDesc& T) { return T.global == 2; }),
                   pl.tiles.end());
  }
  tm.mark("general nets");
  pl.n_global_tiles = 0;
  for (const auto& T : pl.tiles) pl.n_global_tiles += T.global;
  // pipelined tiles (shared-memory window and stage) first, then the rest
  const bool all_slow = getenv("DGR_ALL_SLOW") != nullptr;   // diagnostics: every tile on the slow path
  auto pipelined = [all_slow](const TileDesc& T) {
    return !all_slow && !T.global && T.nbg <= kTargetBundles && T.nb <= kTileBundles && T.ntree <= kPipeTrees &&
           T.nsub <= kPipeSubs && T.nmn <= kTileThreads;
  };
  std::stable_partition(pl.tiles.begin(), pl.tiles.end(), pipelined);
  pl.n_pipe_tiles = 0;
  for (const auto& T : pl.tiles) pl.n_pipe_tiles += pipelined(T);
  if (!getenv("DGR_TILE_SPATIAL")) {   // largest tiles first (LPT): a shorter tail of the last wave of CTAs (+1.5% on ispd19)
    std::stable_sort(pl.tiles.begin(), pl.tiles.begin() + pl.n_pipe_tiles, [](const TileDesc& a, const TileDesc& b) {
      return 4 * a.nbg + (a.nb - a.nbg) > 4 * b.nbg + (b.nb - b.nbg);
    });
  }
  // one (S_H, S_V) tensor-map pair per distinct window shape of the pipelined tiles (TMA box
  // extents <= 256); other tiles take their window by cp.async
  {
    std::map<std::pair<int, int>, int> idx;
    const bool no_tma = getenv("DGR_NO_TMA_WINDOW") != nullptr;
    for (int64_t t = 0; t < (int64_t)pl.tiles.size(); ++t) {
      TileDesc& T = pl.tiles[t];
      T.tmap = -1;
      if (no_tma || t >= pl.n_pipe_tiles || T.ww <= 0 || T.wh <= 0 || win_pitch(T.ww) > 256 || win_pitch(T.wh) > 256) continue;
      auto it = idx.find({T.ww, T.wh});
      if (it == idx.end()) {
        it = idx.emplace(std::make_pair(T.ww, T.wh), (int)pl.tmap_shapes.size()).first;
        pl.tmap_shapes.push_back({T.ww, T.wh});
      }
      T.tmap = it->second;
    }
  }
  return DGR_OK;
}

// ---------------------------------------------------------------------------------------
// TMA tensor maps of the tile windows: 2-D views of S_H ([Y][XP] fp64) and S_V^T ([X][YP] fp64)
// with the window's shape as the box (rows / columns padded to win_pitch), so one copy per field
// lands in the kernel's row-major (column-major) window layout.  cuTensorMapEncodeTiled comes from the driver through the runtime's
// entry-point query (no link against libcuda).
// ---------------------------------------------------------------------------------------
int encode_window_maps(const std::vector<std::pair<int, int>>& shapes, const void* SH, const void* SVT, int X, int Y,
                       unsigned char* out) {
  static PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
  if (!encode) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !fn)
      return -1;
    encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  }
  const cuuint64_t XP = (cuuint64_t)(X + (X & 1)), YP = (cuuint64_t)(Y + (Y & 1));
  for (size_t i = 0; i < shapes.size(); ++i) {
    const cuuint32_t ww = (cuuint32_t)shapes[i].first, wh = (cuuint32_t)shapes[i].second;
    const cuuint32_t es[2] = {1, 1};
    {   // H field: inner dimension x
      const cuuint64_t dims[2] = {XP, (cuuint64_t)Y};
      const cuuint64_t strides[1] = {XP * 8};
      const cuuint32_t box[2] = {(cuuint32_t)win_pitch((int)ww), wh};   // padded rows (columns past X: zeros)
      CUresult r = encode(reinterpret_cast<CUtensorMap*>(out + 256 * i), CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2,
                          const_cast<void*>(SH), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                          CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (r != CUDA_SUCCESS) return (int)r;
    }
    {   // V field: inner dimension y
      const cuuint64_t dims[2] = {YP, (cuuint64_t)X};
      const cuuint64_t strides[1] = {YP * 8};
      const cuuint32_t box[2] = {(cuuint32_t)win_pitch((int)wh), ww};
      CUresult r = encode(reinterpret_cast<CUtensorMap*>(out + 256 * i + 128), CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2,
                          const_cast<void*>(SVT), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                          CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (r != CUDA_SUCCESS) return (int)r;
    }
  }
  return 0;
}

// ---------------------------------------------------------------------------------------
// workspace layout
// ---------------------------------------------------------------------------------------
struct Layout {
  size_t ldesc, tiles, net_gtree, runs, gnet, gtree, gsub, gp_seg_off, gp_tp_off, gseg, gtp, gdq, mnets, tmaps, binfo, pword, sxy, slot_path, wp, mv, pp, nto, wt, mt, vt, q, xbuf, capH, capVT, SH, SVT, dOutH, dOutVT,
      partial, lpart, loss, chosen, tree_choice, route, nsize, nucleus_tmp, DHVC, iscal, ipartial, metrics, total;
  size_t xcount;   // int64 elements in the exchange buffer
  // grid bands (SURVEY §8(e) refinement 2): rank r reduces and scans H rows [r yb, (r+1) yb) and V
  // columns [r xb, (r+1) xb); the row-major H arrays have world * yb rows, the V arrays world * xb
  // columns (padding beyond Y / X), so every rank's band is one contiguous chunk
  int yb = 0, xb = 0;
  size_t gh = 0, gv = 0;   // cells of the H arrays ([world yb][X]) and of the V arrays ([world xb][Y])
};

Layout make_layout(const Plan& pl, int X, int Y, int metric_blocks) {
  Layout L{};
  size_t o = 0;
  auto take = [&](size_t bytes) { size_t r = o; o += (bytes + 255) & ~(size_t)255; return r; };
  // slots: the bundles' 32 per bundle, then the general paths' virtual slots (row f4')
  const size_t bslots = (size_t)pl.nb * 32, slots = bslots + (size_t)pl.n_gpath, ns = pl.sxy.size(),
               nt = (size_t)(pl.tree_hi - pl.tree_lo), nn = (size_t)(pl.net_hi - pl.net_lo), G = (size_t)X * Y;
  L.tiles = take(sizeof(TileDesc) * pl.tiles.size());
  L.gnet = take(sizeof(int2) * pl.gnet.size() + 16);
  L.gtree = take(sizeof(int4) * pl.gtree.size() + 16);
  L.gsub = take(sizeof(GSub) * pl.gsub.size() + 16);
  L.gp_seg_off = take(4 * pl.gp_seg_off.size() + 16);
  L.gp_tp_off = take(4 * pl.gp_tp_off.size() + 16);
  L.gseg = take(8 * pl.gseg.size() + 16);
  L.gtp = take(4 * pl.gtp.size() + 16);
  L.gdq = take(8 * pl.gtree.size() + 16);
  L.mnets = take(4 * pl.mnets.size() + 16);
  L.tmaps = take(256 * pl.tmap_shapes.size() + 256);   // 128-byte CUtensorMaps, (S_H, S_V) per window shape
  L.binfo = take(sizeof(int4) * pl.nb);
  L.pword = take(4 * bslots);
  L.ldesc = take(4 * bslots);
  L.sxy = take(8 * ns + 16);
  L.slot_path = take(4 * slots);
  L.wp = take(4 * slots);
  L.mv = take(8 * slots);
  L.pp = take(4 * slots);   // p of the last forward (read by the next reverse)
  L.nto = take(4 * (nn + 1) + 16);   // +16 B: 16-byte aligned bulk reads may run past the end
  L.net_gtree = take(4 * nn + 16);
  L.runs = take(sizeof(NoiseRun) * pl.runs.size() + 16);
  L.wt = take(4 * nt + 16);
  L.mt = take(4 * nt + 16);
  L.vt = take(4 * nt + 16);
  L.q = take(4 * nt + 16);
  L.yb = (Y + pl.world - 1) / pl.world;
  L.xb = (X + pl.world - 1) / pl.world;
  L.gh = (size_t)pl.world * L.yb * X;
  L.gv = (size_t)pl.world * L.xb * Y;
  L.xcount = L.gh + L.gv + 2;   // dH | dV^T | E[TP], B
  L.xbuf = take(8 * L.xcount);
  L.capH = take(4 * G);
  L.capVT = take(4 * G);
  // S_H [Y][XP] then S_V^T [X][YP] (even pitches, contiguous: one base pointer in the kernels),
  // plus padding for window rows / columns that run one cell past the grid
  const size_t XP = (size_t)(X + (X & 1)), YP = (size_t)(Y + (Y & 1));
  L.SH = take(8 * ((size_t)pl.world * L.yb * XP + (size_t)pl.world * L.xb * YP) + 256);
  L.SVT = L.SH + 8 * (size_t)pl.world * L.yb * XP;
  L.dOutH = take(4 * L.gh);
  L.dOutVT = take(4 * L.gv);
  L.partial = take(8 * (size_t)(X + Y));
  L.lpart = take(8 * (size_t)(X + Y) + 16);   // per-line demand sums, then lsum[2]
  L.loss = take(8 * 4);
  L.chosen = take(nt);
  L.tree_choice = take(4 * nn);
  L.route = take(4 * ns);
  L.nsize = take(4 * ns);
  L.nucleus_tmp = take(4 * slots);
  L.DHVC = take(4 * 3 * G);
  L.iscal = take(8 * 2);
  L.ipartial = take(8 * 3 * (size_t)metric_blocks);
  L.metrics = take(8 * 5);
  L.total = o;
  return L;
}

}  // namespace

namespace dgr {
int set_error(int code, const char* msg) { g_err = msg; return code; }
void clear_error() { g_err.clear(); }
}  // namespace dgr

struct dgr_handle {
  int X = 0, Y = 0;
  int64_t n_nets = 0, n_trees = 0, n_subnets = 0, n_paths = 0;
  Plan plan;
  Layout lay{};
  KParams P{};
  cudaStream_t stream = nullptr;
  int rank = 0, world = 1;
  // the band exchange runs (world > 1, or a one-rank dgr_dist with an NCCL id or a callback: the
  // exchange path exercised on one GPU)
  bool xchg = false;
  ncclComm_t comm = nullptr;
  dgr_allreduce_fn ar_fn = nullptr;   // caller-supplied exchange instead of NCCL (dgr_dist.allreduce)
  void* ar_user = nullptr;
  char* ws = nullptr;
  int64_t ws_bytes = 0;
  int64_t k = 0;
  float t_last = 1.f;
  float beta_last = 0.25f;
  bool have_forward = false;
  // the grids hold the demand events of the forward of iteration k at temperature t_fwd (the
  // last iteration of the previous dgr_step call ran it), so the next call can start from them
  bool fwd_valid = false;
  float t_fwd = 0.f;
  float beta_fwd = 0.f;   // the forward's turning-point demand is folded into the grids with its beta
  // the exchange grids may hold demand events no KG has consumed yet (set before every forward
  // launch, cleared after the KG that reads them): a call that failed part-way leaves it set, and
  // the next call clears the grids instead of adding its events on top of the stale ones
  bool grids_dirty = false;
  double* pinned = nullptr;   // 16 doubles of pinned host memory
  int dev = -1;               // device of the workspace (set at bind); every later call runs on it
  // profiling: a CUDA event after every stage, attributed to that stage
  bool prof = false;
  std::vector<cudaEvent_t> ev;
  std::vector<int> ev_stage;
  size_t ev_used = 0;
};

namespace {
// Makes the handle's device current for the duration of an entry point (the caller's current
// device may differ: launches and stream work must go to the workspace's device) and restores it.
struct DevGuard {
  int prev = -1;
  explicit DevGuard(const dgr_handle* h) {
    if (!h || h->dev < 0) return;
    if (cudaGetDevice(&prev) != cudaSuccess) { prev = -1; return; }
    if (prev != h->dev) cudaSetDevice(h->dev); else prev = -1;
  }
  ~DevGuard() { if (prev >= 0) cudaSetDevice(prev); }
};
// stage -1 opens an interval; stage >= 0 closes the interval since the previous event
int prof_mark(dgr_handle* h, int stage) {
  if (!h->prof) return DGR_OK;
  if (h->ev.size() <= h->ev_used) {
    cudaEvent_t e;
    CUDA_TRY(cudaEventCreate(&e));
    h->ev.push_back(e);
    h->ev_stage.push_back(-1);
  }
  CUDA_TRY(cudaEventRecord(h->ev[h->ev_used], h->stream));
  h->ev_stage[h->ev_used] = stage;
  h->ev_used += 1;
  return DGR_OK;
}
}  // namespace

extern "C" {

const char* dgr_last_error(void) { return g_err.c_str(); }

int dgr_nccl_unique_id(void* out128) {
  g_err.clear();
  if (!out128) return fail(DGR_EINVAL, "out is NULL");
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  ncclUniqueId id;
  NCCL_TRY(ncclGetUniqueId(&id));
  memcpy(out128, &id, sizeof(id));
  return DGR_OK;
}

int dgr_partition(const dgr_forest_desc* desc, int32_t world, int64_t* out) {
  g_err.clear();
  int rc = validate_structure(desc);
  if (rc) return rc;
  if (!out) return fail(DGR_EINVAL, "out is NULL");
  std::vector<int64_t> part;
  if ((rc = partition(desc, world, part))) return rc;
  std::copy(part.begin(), part.end(), out);
  return DGR_OK;
}

// Collectives on the handle's stream, NCCL or the caller's exchange (dgr_dist.allreduce; reduce-scatter
// and all-gather are then expressed through it).  dtype: 0 int64, 1 int32, 2 fp64, 3 fp32.
enum { kI64 = 0, kI32 = 1, kF64 = 2, kF32 = 3 };
static ncclDataType_t nccl_type(int dt) {
  return dt == kI64 ? ncclInt64 : dt == kI32 ? ncclInt32 : dt == kF64 ? ncclFloat64 : ncclFloat32;
}
static size_t dt_bytes(int dt) { return (dt == kI32 || dt == kF32) ? 4 : 8; }
static int live_comm(dgr_handle* h) {
  if (h->xchg && !h->ar_fn && !h->comm) return fail(DGR_ESTATE, "the NCCL communicator was aborted after an error or timeout");
  return DGR_OK;
}
// in-place sum over the ranks
static int allreduce(dgr_handle* h, void* buf, int64_t count, int dtype) {
  if (h->ar_fn) {
    const int r = h->ar_fn(h->ar_user, buf, count, dtype, (void*)h->stream);
    return r ? fail(DGR_ENCCL, "allreduce callback returned %d", r) : DGR_OK;
  }
  NCCL_TRY(ncclAllReduce(buf, buf, (size_t)count, nccl_type(dtype), ncclSum, h->comm, h->stream));
  return DGR_OK;
}
// in place over world chunks of `chunk` elements: this rank's chunk gets the sum of every rank's
// copy of it (the other chunks are left undefined)
static int reduce_scatter(dgr_handle* h, void* buf, int64_t chunk, int dtype) {
  if (h->ar_fn) return allreduce(h, buf, chunk * h->world, dtype);
  NCCL_TRY(ncclReduceScatter(buf, (char*)buf + (size_t)h->rank * chunk * dt_bytes(dtype), (size_t)chunk, nccl_type(dtype),
                             ncclSum, h->comm, h->stream));
  return DGR_OK;
}
// in place over world chunks: every rank's own chunk copied into every rank's buffer
static int all_gather(dgr_handle* h, void* buf, int64_t chunk, int dtype) {
  const size_t cb = (size_t)chunk * dt_bytes(dtype);
  if (h->ar_fn) {   // the other chunks zeroed, then summed: x + 0 + ... + 0 = x exactly
    char* b = (char*)buf;
    if (h->rank > 0) CUDA_TRY(cudaMemsetAsync(b, 0, cb * h->rank, h->stream));
    if (h->rank + 1 < h->world) CUDA_TRY(cudaMemsetAsync(b + cb * (h->rank + 1), 0, cb * (h->world - h->rank - 1), h->stream));
    return allreduce(h, buf, chunk * h->world, dtype);
  }
  NCCL_TRY(ncclAllGather((char*)buf + (size_t)h->rank * cb, buf, (size_t)chunk, nccl_type(dtype), h->comm, h->stream));
  return DGR_OK;
}
static int group_start(dgr_handle* h) { if (!h->ar_fn) NCCL_TRY(ncclGroupStart()); return DGR_OK; }
static int group_end(dgr_handle* h) { if (!h->ar_fn) NCCL_TRY(ncclGroupEnd()); return DGR_OK; }

// Waits for the handle's stream.  With an NCCL communicator: polls, and aborts the communicator
// (ncclCommAbort) on an asynchronous NCCL error or after DGR_NCCL_TIMEOUT_MS (default 300000 ms)
// without completion, so a rank whose peer died returns DGR_ENCCL instead of hanging.
static int wait_stream(dgr_handle* h) {
  if (!h->comm) { CUDA_TRY(cudaStreamSynchronize(h->stream)); return DGR_OK; }
  const char* to = getenv("DGR_NCCL_TIMEOUT_MS");
  const double limit_ms = to ? atof(to) : 300000.0;
  const auto t0 = std::chrono::steady_clock::now();
  for (;;) {
    const cudaError_t e = cudaStreamQuery(h->stream);
    if (e == cudaSuccess) return DGR_OK;
    if (e != cudaErrorNotReady) return fail(DGR_ECUDA, "stream: %s", cudaGetErrorString(e));
    ncclResult_t ar = ncclSuccess;
    ncclCommGetAsyncError(h->comm, &ar);
    const double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    if ((ar != ncclSuccess && ar != ncclInProgress) || ms > limit_ms) {
      ncclCommAbort(h->comm);
      h->comm = nullptr;
      if (ar != ncclSuccess && ar != ncclInProgress)
        return fail(DGR_ENCCL, "NCCL error %s (communicator aborted)", ncclGetErrorString(ar));
      return fail(DGR_ENCCL, "NCCL exchange not complete after %.0f ms (communicator aborted)", ms);
    }
    std::this_thread::sleep_for(std::chrono::microseconds(50));
  }
}

static int dist_args(const dgr_dist* dist, int* rank, int* world) {
  *rank = 0;
  *world = 1;
  if (dist) {
    *rank = dist->rank;
    *world = dist->world;
  }
  if (*world < 1 || *rank < 0 || *rank >= *world) return fail(DGR_EINVAL, "bad rank/world %d/%d", *rank, *world);
  if (*world > 1 && (!dist || (!dist->nccl_unique_id && !dist->allreduce)))
    return fail(DGR_EINVAL, "world > 1 needs an NCCL unique id or an allreduce callback");
  return DGR_OK;
}

int64_t dgr_workspace_size(const dgr_forest_desc* desc, const dgr_dist* dist) {
  g_err.clear();
  int rank, world;
  if (dist_args(dist, &rank, &world)) return 0;
  Plan pl;
  if (make_plan(desc, rank, world, pl)) return 0;
  dgr::KParams tmp{};
  tmp.X = desc->X;
  tmp.Y = desc->Y;
  return (int64_t)make_layout(pl, desc->X, desc->Y, induce_metric_blocks(tmp)).total;
}

int dgr_forest_plan(const dgr_forest_desc* desc, const dgr_dist* dist, void* cuda_stream, dgr_handle** out) {
  g_err.clear();
  if (!out) return fail(DGR_EINVAL, "out is NULL");
  *out = nullptr;
  int rank, world, rc;
  if ((rc = dist_args(dist, &rank, &world))) return rc;
  auto* h = new dgr_handle();
  if ((rc = make_plan(desc, rank, world, h->plan))) { delete h; return rc; }
  h->X = desc->X; h->Y = desc->Y;
  h->n_nets = desc->n_nets; h->n_trees = desc->n_trees; h->n_subnets = desc->n_subnets; h->n_paths = desc->n_paths;
  h->rank = rank; h->world = world;
  h->stream = (cudaStream_t)cuda_stream;
  h->P.X = desc->X; h->P.Y = desc->Y;
  h->lay = make_layout(h->plan, desc->X, desc->Y, induce_metric_blocks(h->P));
  *out = h;
  return DGR_OK;
}

int64_t dgr_handle_workspace_size(dgr_handle* h) {
  g_err.clear();
  if (!h) { fail(DGR_EINVAL, "NULL handle"); return 0; }
  return (int64_t)h->lay.total;
}

int dgr_forest_load(const dgr_forest_desc* desc, const dgr_dist* dist, void* dev_workspace, int64_t workspace_bytes,
                    void* cuda_stream, dgr_handle** out) {
  g_err.clear();
  if (!out) return fail(DGR_EINVAL, "out is NULL");
  *out = nullptr;
  dgr_handle* h = nullptr;
  int rc;
  if ((rc = dgr_forest_plan(desc, dist, cuda_stream, &h))) return rc;
  if ((rc = dgr_bind_workspace(h, desc, dist, dev_workspace, workspace_bytes))) {
    const std::string msg = g_err;
    dgr_free(h);
    g_err = msg;
    return rc;
  }
  *out = h;
  return DGR_OK;
}

int dgr_bind_workspace(dgr_handle* h, const dgr_forest_desc* desc, const dgr_dist* dist, void* dev_workspace,
                       int64_t workspace_bytes) {
  g_err.clear();
  if (!h || !desc) return fail(DGR_EINVAL, "NULL handle or desc");
  if (h->ws) return fail(DGR_ESTATE, "the handle already has a workspace");
  if (desc->X != h->X || desc->Y != h->Y || desc->n_nets != h->n_nets || desc->n_trees != h->n_trees ||
      desc->n_subnets != h->n_subnets || desc->n_paths != h->n_paths)
    return fail(DGR_EINVAL, "desc does not describe the planned forest");
  int rank, world, rc;
  if ((rc = dist_args(dist, &rank, &world))) return rc;
  if (rank != h->rank || world != h->world) return fail(DGR_EINVAL, "dist differs from the one planned with");
  const Plan& pl = h->plan;
  KParams& P = h->P;
  const Layout& L = h->lay;
  if (!dev_workspace || workspace_bytes < (int64_t)L.total)
    return fail(DGR_ENOMEM, "workspace of %lld bytes < %zu needed", (long long)workspace_bytes, L.total);
  if (((uintptr_t)dev_workspace) & 255) return fail(DGR_EINVAL, "workspace not 256-byte aligned");
  {
    cudaPointerAttributes pa{};
    if (cudaPointerGetAttributes(&pa, dev_workspace) != cudaSuccess || pa.type != cudaMemoryTypeDevice) {
      cudaGetLastError();
      return fail(DGR_EINVAL, "workspace is not device memory");
    }
    h->dev = pa.device;
  }
  DevGuard dg(h);
  char* ws = (char*)dev_workspace;
  P.nb = pl.nb;
  P.ntiles = (int32_t)pl.n_pipe_tiles;
  P.tiles = (const TileDesc*)(ws + L.tiles);
  P.ntiles_slow = (int32_t)(pl.tiles.size() - pl.n_pipe_tiles);
  P.tiles_slow = P.tiles + pl.n_pipe_tiles;
  P.XP = desc->X + (desc->X & 1);
  if (const char* sk = getenv("DGR_DEBUG_SKIP")) P.skip = atoi(sk);   // timing experiments only
  P.pf = 2;   // L2 prefetch of the trees' Adam moments only (+0.4%; of the slots' state too: no gain, A/B)
  if (const char* e = getenv("DGR_PF")) P.pf = atoi(e);
  P.YP = desc->Y + (desc->Y & 1);
  P.n_nets_l = (int32_t)(pl.net_hi - pl.net_lo);
  P.path_base = pl.path_lo;
  P.tree_base = pl.tree_lo;
  P.nid_base = pl.nid_base;
  P.seed = desc->seed;
  P.mnets = (const uint32_t*)(ws + L.mnets);
  P.ngen = (int32_t)pl.gnet.size();
  P.ngen_blocks = (P.ngen + kGenWarps - 1) / kGenWarps;
  P.ngsub = (int32_t)pl.gsub.size();
  P.gnet = (const int2*)(ws + L.gnet);
  P.gtree = (const int4*)(ws + L.gtree);
  P.gsub = (const GSub*)(ws + L.gsub);
  P.gp_seg_off = (const int32_t*)(ws + L.gp_seg_off);
  P.gp_tp_off = (const int32_t*)(ws + L.gp_tp_off);
  P.gseg = (const short4*)(ws + L.gseg);
  P.gtp = (const short2*)(ws + L.gtp);
  P.gdq = (long long*)(ws + L.gdq);
  P.tmaps = (const unsigned char*)(ws + L.tmaps);
  for (int r = 0; r < 10; ++r) {   // Philox4x32-10 round keys of the seed
    P.rk[2 * r] = (uint32_t)desc->seed + (uint32_t)r * 0x9E3779B9u;
    P.rk[2 * r + 1] = (uint32_t)(desc->seed >> 32) + (uint32_t)r * 0xBB67AE85u;
  }
  P.binfo = (const int4*)(ws + L.binfo);
  P.pword = (const uint32_t*)(ws + L.pword);
  P.ldesc = (const uint32_t*)(ws + L.ldesc);
  P.sxy = (const short4*)(ws + L.sxy);
  P.slot_path = (const int32_t*)(ws + L.slot_path);
  P.wp = (float*)(ws + L.wp); P.mv = (float2*)(ws + L.mv);
  P.pp = (float*)(ws + L.pp);
  P.net_tree_off = (const int32_t*)(ws + L.nto);
  P.net_gtree = (const int32_t*)(ws + L.net_gtree);
  P.perm_id = 1;
  for (size_t i = 0; i < pl.perm.size() && P.perm_id; ++i) P.perm_id = pl.perm[i] == (int64_t)i;
  P.runs = (const NoiseRun*)(ws + L.runs);
  P.wt = (float*)(ws + L.wt); P.mt = (float*)(ws + L.mt); P.vt = (float*)(ws + L.vt); P.q = (float*)(ws + L.q);
  const size_t G = (size_t)desc->X * desc->Y;
  P.dH = (long long*)(ws + L.xbuf);
  P.dVT = P.dH + L.gh;
  P.acc = P.dVT + L.gv;
  // the rank's KG lines (its grid bands; all lines on one GPU)
  P.kg_h0 = std::min(desc->Y, rank * L.yb); P.kg_h1 = std::min(desc->Y, (rank + 1) * L.yb);
  P.kg_v0 = std::min(desc->X, rank * L.xb); P.kg_v1 = std::min(desc->X, (rank + 1) * L.xb);
  P.capH = (const float*)(ws + L.capH);
  P.capVT = (const float*)(ws + L.capVT);
  P.SH = (double*)(ws + L.SH); P.SVT = (double*)(ws + L.SVT);
  P.dOutH = (float*)(ws + L.dOutH); P.dOutVT = (float*)(ws + L.dOutVT);
  P.partial = (double*)(ws + L.partial);
  P.lpart = (long long*)(ws + L.lpart);
  P.lsum = P.lpart + (desc->X + desc->Y);
  P.loss = (double*)(ws + L.loss);
  P.chosen = (uint8_t*)(ws + L.chosen);
  P.tree_choice = (int32_t*)(ws + L.tree_choice);
  P.route = (int32_t*)(ws + L.route);
  P.nsize = (int32_t*)(ws + L.nsize);
  P.nucleus_tmp = (int32_t*)(ws + L.nucleus_tmp);
  P.DH = (int32_t*)(ws + L.DHVC);
  P.DV = P.DH + G;
  P.VC = P.DV + G;
  P.iscal = (long long*)(ws + L.iscal);
  P.ipartial = (double*)(ws + L.ipartial);
  P.metrics = (double*)(ws + L.metrics);

  auto cleanup = [&](int code) {   // back to the planned state
    if (h->pinned) { cudaFreeHost(h->pinned); h->pinned = nullptr; }
    h->P = KParams{};
    h->P.X = h->X; h->P.Y = h->Y;
    return code;
  };
  cudaStream_t s = h->stream;
  PhaseTimer tm;
  if (prepare_kernels() != 0) return cleanup(fail(DGR_ECUDA, "cudaFuncSetAttribute (tile kernel shared memory) failed"));
  tm.mark("bind: prepare kernels");
  if (cudaMemsetAsync(ws, 0, L.total, s) != cudaSuccess) return cleanup(fail(DGR_ECUDA, "memset workspace failed"));
  // host-side staging of the encoded shard, packed into pinned memory, then one copy per region
  const size_t slots = (size_t)pl.nb * 32 + (size_t)pl.n_gpath;   // bundle slots, then general (virtual) slots
  const size_t nt = (size_t)(pl.tree_hi - pl.tree_lo);
  struct Region { size_t off, bytes; const void* src; };   // src == nullptr: filled in place below
  std::vector<Region> regs = {
      {L.tiles, sizeof(TileDesc) * pl.tiles.size(), pl.tiles.data()},
      {L.mnets, 4 * pl.mnets.size(), pl.mnets.data()},
      {L.binfo, sizeof(int4) * pl.nb, pl.binfo.data()},
      {L.pword, 4 * (size_t)pl.nb * 32, pl.pword.data()},
      {L.sxy, 8 * pl.sxy.size(), pl.sxy.data()},
      {L.wp, 4 * slots, nullptr},
      {L.pp, 4 * slots, nullptr},
      {L.slot_path, 4 * slots, pl.slot_path.data()},
      {L.nto, 4 * pl.net_tree_off.size(), pl.net_tree_off.data()},
      {L.wt, 4 * nt, nullptr},   // plan (tile) order of the trees
      {L.q, 4 * nt, nullptr},
      {L.capH, 4 * G, desc->cap_h},
      {L.capVT, 4 * G, nullptr},
      {L.tmaps, 256 * pl.tmap_shapes.size(), nullptr},
      {L.gnet, sizeof(int2) * pl.gnet.size(), pl.gnet.data()},
      {L.gtree, sizeof(int4) * pl.gtree.size(), pl.gtree.data()},
      {L.gsub, sizeof(GSub) * pl.gsub.size(), pl.gsub.data()},
      {L.gp_seg_off, 4 * pl.gp_seg_off.size(), pl.gp_seg_off.data()},
      {L.gp_tp_off, 4 * pl.gp_tp_off.size(), pl.gp_tp_off.data()},
      {L.gseg, 8 * pl.gseg.size(), pl.gseg.data()},
      {L.gtp, 4 * pl.gtp.size(), pl.gtp.data()},
      {L.net_gtree, 4 * pl.net_gtree.size(), pl.net_gtree.data()},
      {L.runs, sizeof(NoiseRun) * pl.runs.size(), pl.runs.data()},
      {L.ldesc, 4 * (size_t)pl.nb * 32, pl.ldesc.data()}};   // (regions 5, 6, 9, 10, 12, 13 are filled in place below)
  std::vector<size_t> at(regs.size() + 1, 0);
  for (size_t i = 0; i < regs.size(); ++i) at[i + 1] = at[i] + ((regs[i].bytes + 255) & ~(size_t)255);
  std::lock_guard<std::mutex> lock(g_pin.m);
  char* pin = g_pin.get(at.back());
  if (!pin) return cleanup(fail(DGR_ENOMEM, "cudaHostAlloc of %zu staging bytes failed", at.back()));
  float* wslots = reinterpret_cast<float*>(pin + at[5]);
  float* pslots = reinterpret_cast<float*>(pin + at[6]);
  float* qs = reinterpret_cast<float*>(pin + at[10]);
  float* wts = reinterpret_cast<float*>(pin + at[9]);
#pragma omp parallel for schedule(static)
  for (size_t j = 0; j < nt; ++j) {
    wts[j] = desc->w_tree0[pl.tree_lo + pl.tperm[j]];
    qs[j] = 1.f;   // q of a net's lone tree stays 1 (never rewritten)
  }
  float* capVT = reinterpret_cast<float*>(pin + at[12]);
#pragma omp parallel for schedule(static)
  for (size_t sl = 0; sl < slots; ++sl) {
    const bool v = pl.slot_path[sl] >= 0;
    wslots[sl] = v ? desc->w_path0[pl.path_lo + pl.slot_path[sl]] : 0.f;
    pslots[sl] = v ? 1.f : 0.f;   // p of a lone straight candidate (never rewritten by the pipelined kernel)
  }
  // tensor maps of the tile windows over this workspace's S_H ([Y][XP]) and S_V ([X][YP]) (fp64)
  if (!pl.tmap_shapes.empty()) {
    unsigned char* tm = reinterpret_cast<unsigned char*>(pin + at[13]);
    const int rc = encode_window_maps(pl.tmap_shapes, (const void*)P.SH, (const void*)P.SVT, desc->X, desc->Y, tm);
    if (rc) return cleanup(fail(DGR_ECUDA, "cuTensorMapEncodeTiled failed (%d)", rc));
  }
#pragma omp parallel for schedule(static)
  for (int y = 0; y < desc->Y; ++y)
    for (int x = 0; x < desc->X; ++x) capVT[(size_t)x * desc->Y + y] = desc->cap_v[(size_t)y * desc->X + x];
  tm.mark("bind: host staging (in place)");
  // stage region i and start its upload, so that the DMA of region i overlaps the staging of i+1
  cudaError_t e = cudaSuccess;
  for (size_t i = 0; i < regs.size() && e == cudaSuccess; ++i) {
    if (!regs[i].bytes) continue;
    if (regs[i].src) par_copy(pin + at[i], regs[i].src, regs[i].bytes);
    e = cudaMemcpyAsync(ws + regs[i].off, pin + at[i], regs[i].bytes, cudaMemcpyHostToDevice, s);
  }
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  tm.mark("bind: staging + upload");
  if (e != cudaSuccess) return cleanup(fail(DGR_ECUDA, "upload: %s", cudaGetErrorString(e)));
  if (cudaMallocHost(&h->pinned, 16 * sizeof(double)) != cudaSuccess) return cleanup(fail(DGR_ECUDA, "cudaMallocHost failed"));
  h->xchg = dist && (world > 1 || dist->nccl_unique_id || dist->allreduce);
  if (h->xchg && dist->allreduce) {
    h->ar_fn = dist->allreduce;
    h->ar_user = dist->allreduce_user;
  } else if (h->xchg) {
    ncclUniqueId id;
    memcpy(&id, dist->nccl_unique_id, sizeof(id));
    ncclResult_t r = ncclCommInitRank(&h->comm, world, id, rank);
    if (r != ncclSuccess) return cleanup(fail(DGR_ENCCL, "ncclCommInitRank: %s", ncclGetErrorString(r)));
  }
  h->ws = ws;
  h->ws_bytes = workspace_bytes;
  return DGR_OK;
}

static int step_impl(dgr_handle* h, int32_t iters, float temperature, float lr, const dgr_weights* w, dgr_loss* last,
                     double* loss_async);

int dgr_step(dgr_handle* h, int32_t iters, float temperature, float lr, const dgr_weights* w, dgr_loss* last) {
  return step_impl(h, iters, temperature, lr, w, last, nullptr);
}

int dgr_step_async(dgr_handle* h, int32_t iters, float temperature, float lr, const dgr_weights* w,
                   double* loss_out) {
  g_err.clear();
  if (!loss_out) return fail(DGR_EINVAL, "NULL loss_out");
  return step_impl(h, iters, temperature, lr, w, nullptr, loss_out);
}

int dgr_sync(dgr_handle* h) {
  g_err.clear();
  DevGuard dg(h);
  if (!h) return fail(DGR_EINVAL, "NULL handle");
  return wait_stream(h);
}

static int step_impl(dgr_handle* h, int32_t iters, float temperature, float lr, const dgr_weights* w, dgr_loss* last,
                     double* loss_async) {
  g_err.clear();
  DevGuard dg(h);
  if (!h || !w) return fail(DGR_EINVAL, "NULL handle or weights");
  if (!h->ws) return fail(DGR_ESTATE, "no workspace bound (dgr_bind_workspace)");
  if (iters < 0) return fail(DGR_EINVAL, "iters < 0");
  if (!(temperature > 0.f) || !std::isfinite(temperature)) return fail(DGR_EINVAL, "temperature must be > 0");
  if (w->f_kind < 0 || w->f_kind > 4) return fail(DGR_EINVAL, "f_kind must be 0..4 (sigmoid, ReLU, LeakyReLU, exp, CELU)");
  if ((w->f_kind == 0 || w->f_kind == 3 || w->f_kind == 4) && !(w->f_slope > 0.f))
    return fail(DGR_EINVAL, "f_slope must be > 0 for sigmoid / exp / CELU");
  if (int rc0 = live_comm(h)) return rc0;
  KParams& P = h->P;
  // the loss goes straight from kg_loss_kernel into a pinned (device-accessible) host buffer: the
  // caller's (dgr_step_async) or the handle's (dgr_step); a pageable buffer gets a copy after it
  double* loss_dev = nullptr;
  {
    double* want = loss_async ? loss_async : (last ? h->pinned : nullptr);
    cudaPointerAttributes at{};
    if (want && cudaPointerGetAttributes(&at, want) == cudaSuccess && at.type == cudaMemoryTypeHost && at.devicePointer)
      loss_dev = static_cast<double*>(at.devicePointer);
    cudaGetLastError();   // a pageable pointer may leave an error code behind
  }
  StepArgs a{};
  a.inv_t = 1.f / temperature;
  a.a_wl = w->a_wl; a.a_via = w->a_via; a.a_of = w->a_of; a.beta = w->beta_via;
  a.sqrt_l = std::sqrt(w->n_layers);
  a.f_slope = w->f_slope; a.f_kind = w->f_kind;
  a.beta_q = (double)w->beta_via * kGridBeta;
  a.beta_d = (double)a.beta;
  a.a_wl_d = (double)a.a_wl;
  a.via_d = (double)a.a_via * (double)a.sqrt_l;
  a.beta_exact = std::nearbyint(a.beta_q) == a.beta_q && std::fabs(a.beta_q) < 9.0e15;
  a.beta_qi = a.beta_exact ? (long long)a.beta_q : 0;
  const size_t xbytes = 8 * h->lay.xcount;
  (void)xbytes;
  cudaStream_t s = h->stream;
  auto adam_args = [&](int64_t k) {
    const double step = (double)(k + 1);
    a.lr_over_bc1 = (float)(lr / (1.0 - std::pow(0.9, step)));
    a.inv_sqrt_bc2 = (float)(1.0 / std::sqrt(1.0 - std::pow(0.999, step)));
  };
  int rc;
  // forward of iteration k (q, p, demand events of the current logits at this temperature),
  // unless the previous call left exactly that forward in the grids
  a.k = h->k;
  a.k_next = h->k;
  a.store_d = 0;
  adam_args(h->k);
  if ((rc = prof_mark(h, -1))) return rc;
  if (!(h->fwd_valid && h->t_fwd == temperature && h->beta_fwd == w->beta_via)) {
    // KG clears the event grids in place after reading them; stale events of a forward at another
    // temperature are cleared here
    if (h->grids_dirty) CUDA_TRY(cudaMemsetAsync(P.dH, 0, 8 * h->lay.xcount, s));   // dH | dV^T | E[WL], E[TP]
    h->grids_dirty = true;
    launch_tiles(P, a, kForwardOnly, s);
    if ((rc = prof_mark(h, 0))) return rc;
  }
  h->fwd_valid = false;
  const int n = iters == 0 ? 1 : iters;
  for (int it = 0; it < n; ++it) {
    const bool last = (it == n - 1);
    a.k = h->k;
    a.k_next = h->k + 1;
    a.store_d = last;
    adam_args(h->k);
    const Layout& Lay = h->lay;
    if (h->xchg) {
      // the forward's events reduced into each rank's grid bands (SURVEY §8(e) refinement 2), the
      // counters summed; the other ranks' bands cleared for the next forward (KG clears its own)
      const int r = h->rank;
      const size_t hb = (size_t)Lay.yb * h->X, vb = (size_t)Lay.xb * h->Y;
      if ((rc = group_start(h)) || (rc = reduce_scatter(h, P.dH, (int64_t)hb, kI64)) ||
          (rc = reduce_scatter(h, P.dVT, (int64_t)vb, kI64)) || (rc = allreduce(h, P.acc, 2, kI64)) || (rc = group_end(h)))
        return rc;
      if (r > 0) CUDA_TRY(cudaMemsetAsync(P.dH, 0, 8 * hb * r, s));
      if (r + 1 < h->world) CUDA_TRY(cudaMemsetAsync(P.dH + hb * (r + 1), 0, 8 * hb * (h->world - r - 1), s));
      if (r > 0) CUDA_TRY(cudaMemsetAsync(P.dVT, 0, 8 * vb * r, s));
      if (r + 1 < h->world) CUDA_TRY(cudaMemsetAsync(P.dVT + vb * (r + 1), 0, 8 * vb * (h->world - r - 1), s));
      if (last) {   // the loss sums every line's partial: the other bands' lines enter as zeros
        CUDA_TRY(cudaMemsetAsync(P.partial, 0, 8 * (size_t)(h->X + h->Y), s));
        CUDA_TRY(cudaMemsetAsync(P.lpart, 0, 8 * (size_t)(h->X + h->Y), s));
      }
      if ((rc = prof_mark(h, 1))) return rc;
    }
    launch_kg(P, a, s);   // this rank's bands (every line on one GPU)
    h->grids_dirty = false;
    if ((rc = prof_mark(h, 2))) return rc;
    if (h->xchg) {
      // the prefix sums S of every band to every rank (each rank's tiles read any of them); in the
      // last iteration also the loss partials and the demand of get_demand
      const size_t XP = (size_t)P.XP, YP = (size_t)P.YP;
      if ((rc = group_start(h)) || (rc = all_gather(h, P.SH, (int64_t)(Lay.yb * XP), kF64)) ||
          (rc = all_gather(h, P.SVT, (int64_t)(Lay.xb * YP), kF64)))
        return rc;
      if (last && ((rc = allreduce(h, P.partial, h->X + h->Y, kF64)) || (rc = allreduce(h, P.lpart, h->X + h->Y, kI64)) ||
                   (rc = all_gather(h, P.dOutH, (int64_t)Lay.yb * h->X, kF32)) ||
                   (rc = all_gather(h, P.dOutVT, (int64_t)Lay.xb * h->Y, kF32))))
        return rc;
      if ((rc = group_end(h))) return rc;
      if ((rc = prof_mark(h, 1))) return rc;
    }
    if (last) {   // the reported loss of this call's last forward
      KParams PL = P;
      PL.loss_host = loss_dev;
      launch_kg_loss(PL, a, s);
      if ((rc = prof_mark(h, 5))) return rc;
    }
    if (iters > 0) {
      // reverse of iteration k + forward of k+1 (also after the last iteration: the next call
      // at the same temperature starts from it)
      h->grids_dirty = true;
      launch_tiles(P, a, kReverseForward, s);
      h->k += 1;
      if ((rc = prof_mark(h, 3))) return rc;
    }
  }
  if (iters > 0) {
    h->fwd_valid = true;
    h->t_fwd = temperature;
    h->beta_fwd = w->beta_via;
  }
  CUDA_TRY(cudaGetLastError());
  if ((P.skip & 256) && getenv("DGR_PROF_OUT")) {   // diagnostics: per-tile phase clocks of the last KBF
    CUDA_TRY(cudaStreamSynchronize(s));
    std::vector<long long> buf(8 * (size_t)P.ntiles);
    CUDA_TRY((cudaError_t)read_tile_prof(buf.data(), P.ntiles));
    if (FILE* f = fopen(getenv("DGR_PROF_OUT"), "wb")) {
      fwrite(buf.data(), 8, buf.size(), f);
      fclose(f);
    }
  }
  h->t_last = temperature;
  h->beta_last = w->beta_via;
  h->have_forward = true;
  if (loss_async && !loss_dev)   // stream-ordered read of this call's loss; no host synchronisation
    CUDA_TRY(cudaMemcpyAsync(loss_async, P.loss, 4 * sizeof(double), cudaMemcpyDeviceToHost, s));
  if (last) {
    if (!loss_dev) CUDA_TRY(cudaMemcpyAsync(h->pinned, P.loss, 4 * sizeof(double), cudaMemcpyDeviceToHost, s));
    if (int rc_ = wait_stream(h)) return rc_;
    last->total = h->pinned[0];
    last->wl = h->pinned[1];
    last->via = h->pinned[2];
    last->overflow = h->pinned[3];
  }
  return DGR_OK;
}

int dgr_get_demand(dgr_handle* h, float* d_h, float* d_v) {
  g_err.clear();
  DevGuard dg(h);
  if (!h || !d_h || !d_v) return fail(DGR_EINVAL, "NULL argument");
  if (!h->ws) return fail(DGR_ESTATE, "no workspace bound (dgr_bind_workspace)");
  if (!h->have_forward) return fail(DGR_ESTATE, "no forward has run yet");
  const size_t G = (size_t)h->X * h->Y;
  std::vector<float> vt(G);
  CUDA_TRY(cudaMemcpyAsync(d_h, h->P.dOutH, 4 * G, cudaMemcpyDeviceToHost, h->stream));
  CUDA_TRY(cudaMemcpyAsync(vt.data(), h->P.dOutVT, 4 * G, cudaMemcpyDeviceToHost, h->stream));
  if (int rc_ = wait_stream(h)) return rc_;
  for (int x = 0; x < h->X; ++x)
    for (int y = 0; y < h->Y; ++y) d_v[(size_t)y * h->X + x] = vt[(size_t)x * h->Y + y];
  return DGR_OK;
}

int dgr_get_logits(dgr_handle* h, float* w_tree, float* w_path) {
  g_err.clear();
  DevGuard dg(h);
  if (!h) return fail(DGR_EINVAL, "NULL handle");
  if (!h->ws) return fail(DGR_ESTATE, "no workspace bound (dgr_bind_workspace)");
  const Plan& pl = h->plan;
  if (w_path) {
    std::vector<float> slots((size_t)pl.nb * 32 + (size_t)pl.n_gpath);
    CUDA_TRY(cudaMemcpyAsync(slots.data(), h->P.wp, 4 * slots.size(), cudaMemcpyDeviceToHost, h->stream));
    if (int rc_ = wait_stream(h)) return rc_;
    for (size_t sl = 0; sl < slots.size(); ++sl)
      if (pl.slot_path[sl] >= 0) w_path[pl.path_lo + pl.slot_path[sl]] = slots[sl];
  }
  if (w_tree) {   // the device holds the trees in plan order (tperm: plan order -> local CSR)
    std::vector<float> wt((size_t)(pl.tree_hi - pl.tree_lo));
    CUDA_TRY(cudaMemcpyAsync(wt.data(), h->P.wt, 4 * wt.size(), cudaMemcpyDeviceToHost, h->stream));
    if (int rc_ = wait_stream(h)) return rc_;
    for (size_t j = 0; j < wt.size(); ++j) w_tree[pl.tree_lo + pl.tperm[j]] = wt[j];
  }
  return DGR_OK;
}

int dgr_induce(dgr_handle* h, float top_p, int32_t* tree_choice, int32_t* route, int64_t* nucleus_off,
               int32_t* nucleus, int32_t* D_h, int32_t* D_v, double metrics[5]) {
  g_err.clear();
  DevGuard dg(h);
  if (!h || !tree_choice || !route || !nucleus_off || !nucleus || !D_h || !D_v || !metrics)
    return fail(DGR_EINVAL, "NULL argument");
  if (!h->ws) return fail(DGR_ESTATE, "no workspace bound (dgr_bind_workspace)");
  if (!(top_p >= 0.f) || !std::isfinite(top_p)) return fail(DGR_EINVAL, "top_p must be finite and >= 0");
  KParams& P = h->P;
  const Plan& pl = h->plan;
  cudaStream_t s = h->stream;
  const size_t G = (size_t)h->X * h->Y;
  CUDA_TRY(cudaMemsetAsync(P.DH, 0, 4 * 3 * G, s));
  CUDA_TRY(cudaMemsetAsync(P.iscal, 0, 16, s));
  launch_induce(P, h->t_last, top_p, h->beta_last, s);
  if (h->xchg) {
    int rc;
    if ((rc = allreduce(h, P.DH, (int64_t)(3 * G), 1))) return rc;
    if ((rc = allreduce(h, P.iscal, 2, 0))) return rc;
  }
  launch_induce_metrics(P, h->beta_last, s);
  CUDA_TRY(cudaGetLastError());
  const int64_t nn = pl.net_hi - pl.net_lo, ns = pl.sub_hi - pl.sub_lo;
  std::vector<int32_t> tc(nn), rt(ns), nsz(ns), nuc((size_t)pl.nb * 32 + (size_t)pl.n_gpath);
  CUDA_TRY(cudaMemcpyAsync(tc.data(), P.tree_choice, 4 * nn, cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaMemcpyAsync(rt.data(), P.route, 4 * ns, cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaMemcpyAsync(nsz.data(), P.nsize, 4 * ns, cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaMemcpyAsync(nuc.data(), P.nucleus_tmp, 4 * nuc.size(), cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaMemcpyAsync(D_h, P.DH, 4 * G, cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaMemcpyAsync(D_v, P.DV, 4 * G, cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaMemcpyAsync(h->pinned, P.metrics, 5 * sizeof(double), cudaMemcpyDeviceToHost, s));
  if (int rc_ = wait_stream(h)) return rc_;
  for (int i = 0; i < 5; ++i) metrics[i] = h->pinned[i];
  if (h->world > 1) {
    std::fill(tree_choice, tree_choice + h->n_nets, -1);
    std::fill(route, route + h->n_subnets, -1);
  }
  for (int64_t pn = 0; pn < nn; ++pn) tree_choice[pl.net_lo + pl.perm[pn]] = tc[pn];   // plan order -> CSR
  // route / nsize come in kernel sub-net order; nucleus_tmp holds each sub-net's nucleus in rank
  // order from its first candidate's slot on
  std::vector<int32_t> nsz_csr(ns);
  for (int64_t ks = 0; ks < ns; ++ks) {
    route[pl.sub_lo + pl.ksub_csr[ks]] = rt[ks];
    nsz_csr[pl.ksub_csr[ks]] = nsz[ks];
  }
  int64_t pos = 0;
  nucleus_off[0] = 0;
  for (int64_t sg = 0; sg < h->n_subnets; ++sg) {
    if (sg >= pl.sub_lo && sg < pl.sub_hi) {
      const int64_t ls = sg - pl.sub_lo;
      for (int r = 0; r < nsz_csr[ls]; ++r) nucleus[pos++] = nuc[(size_t)pl.sub_first_slot[ls] + r];
    }
    nucleus_off[sg + 1] = pos;
  }
  return DGR_OK;
}

int dgr_get_info(dgr_handle* h, int64_t info[12]) {
  g_err.clear();
  if (!h || !info) return fail(DGR_EINVAL, "NULL argument");
  info[0] = h->k; info[1] = h->plan.net_lo; info[2] = h->plan.net_hi; info[3] = h->plan.nb;
  info[4] = (int64_t)h->plan.nb * 32; info[5] = (int64_t)h->lay.total; info[6] = h->world; info[7] = h->rank;
  info[8] = (int64_t)h->plan.tiles.size(); info[9] = h->plan.n_global_tiles; info[10] = h->plan.n_pipe_tiles;
  info[11] = h->plan.n_gpath;
  return DGR_OK;
}

int dgr_plan_info(const dgr_forest_desc* desc, const dgr_dist* dist, int64_t out[8]) {
  g_err.clear();
  if (!out) return fail(DGR_EINVAL, "out is NULL");
  int rank, world, rc;
  if ((rc = dist_args(dist, &rank, &world))) return rc;
  Plan pl;
  if ((rc = make_plan(desc, rank, world, pl))) return rc;
  int64_t maxw = 0, gpaths = 0;
  for (const auto& T : pl.tiles) {
    maxw = std::max<int64_t>(maxw, (int64_t)T.ww * T.wh);
    if (T.global)
      for (int b = T.b0; b < T.b0 + T.nb; ++b) gpaths += pl.binfo[b].w & 0xff;
  }
  dgr::KParams tmp{};
  tmp.X = desc->X;
  tmp.Y = desc->Y;
  out[0] = (int64_t)pl.tiles.size(); out[1] = pl.n_global_tiles; out[2] = pl.nb; out[3] = (int64_t)pl.nb * 32;
  out[4] = (int64_t)make_layout(pl, desc->X, desc->Y, induce_metric_blocks(tmp)).total;
  out[5] = pl.path_hi - pl.path_lo; out[6] = gpaths; out[7] = maxw;
  return DGR_OK;
}

int dgr_profile(dgr_handle* h, int32_t enable) {
  g_err.clear();
  DevGuard dg(h);
  if (!h) return fail(DGR_EINVAL, "NULL handle");
  h->prof = enable != 0;
  h->ev_used = 0;
  return DGR_OK;
}

int dgr_profile_read(dgr_handle* h, double ms[8], int64_t launches[8]) {
  g_err.clear();
  DevGuard dg(h);
  if (!h || !ms || !launches) return fail(DGR_EINVAL, "NULL argument");
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  for (int i = 0; i < 8; ++i) { ms[i] = 0.0; launches[i] = 0; }
  for (size_t i = 1; i < h->ev_used; ++i) {
    const int st = h->ev_stage[i];
    if (st < 0 || st >= 8) continue;
    float t = 0.f;
    CUDA_TRY(cudaEventElapsedTime(&t, h->ev[i - 1], h->ev[i]));
    ms[st] += t;
    launches[st] += 1;
  }
  return DGR_OK;
}

int dgr_free(dgr_handle* h) {
  g_err.clear();
  DevGuard dg(h);
  if (!h) return DGR_OK;
  if (h->stream) cudaStreamSynchronize(h->stream);
  for (auto e : h->ev) cudaEventDestroy(e);
  if (h->comm) ncclCommDestroy(h->comm);
  if (h->pinned) cudaFreeHost(h->pinned);
  delete h;
  return DGR_OK;
}

}  // extern "C"
