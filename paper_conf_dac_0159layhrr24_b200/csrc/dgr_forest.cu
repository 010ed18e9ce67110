// dgr_forest.cu — row f1: net-parallel construction of the routing DAG forest on the GPU
// (§4.2; "a process that can be efficiently accelerated by net-level
// parallelism").  Readings: Q17 tree candidates, Q14 path patterns,
// Q8 initial logits.
//
//   kb_trees   one thread per net: Prim MST from pin 0 (ties to the lowest index); the second
//              candidate = iterated 1-Steiner on the Hanan grid (<= 8 pins) or Prim from the last
//              pin (ties to the highest index), dropped if its edge set equals the first; canonical
//              sub-nets into per-net scratch; per-net counts of trees / sub-nets / paths /
//              segments / turning points
//   scans      exclusive prefix sums of the five count arrays (three-phase, int64)
//   kb_fill    one thread per net: the CSR arrays of its trees, sub-nets and path candidates
//   kb_logits  w0 ~ U[0,1) per tree and path (splitmix64 counter hash)
//
// The result is bit-identical to the host generator (forestgen) and to the f1 oracle
// (oracle/forest_oracle.c) for the same pins.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "dgr.h"
#include "dgr_internal.h"

namespace {

int ffail(int code, const char* fmt, ...) {   // reported through dgr_last_error
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  return dgr::set_error(code, buf);
}

constexpr int kMaxPins = 32;
constexpr int kMaxPts = 64;          // pins + Steiner points
constexpr int kSubPerPin = 3;        // sub-net scratch per pin (two trees: < 3 k edges)
constexpr int kScanBlock = 1024;

struct Pt { int x, y; };

__device__ __forceinline__ int manh(Pt a, Pt b) { return abs(a.x - b.x) + abs(a.y - b.y); }

// Prim over pts[0..n) from root; tie_low: lowest index among equal keys, else highest.
// Edges (parent, child) in joining order; returns the length.
__device__ int prim(const Pt* pts, int n, int root, bool tie_low, unsigned char (*edges)[2], int* n_edges) {
  int dist[kMaxPts];
  signed char par[kMaxPts];
  unsigned long long in = 0ull;
  for (int i = 0; i < n; ++i) { dist[i] = 1 << 30; par[i] = -1; }
  dist[root] = 0;
  int total = 0, ne = 0;
  for (int it = 0; it < n; ++it) {
    int best = -1;
    for (int i = 0; i < n; ++i) {
      if ((in >> i) & 1ull) continue;
      if (best < 0 || dist[i] < dist[best] || (dist[i] == dist[best] && !tie_low)) best = i;
    }
    in |= 1ull << best;
    total += dist[best];
    if (par[best] >= 0) {
      if (edges) { edges[ne][0] = (unsigned char)par[best]; edges[ne][1] = (unsigned char)best; }
      ++ne;
    }
    for (int i = 0; i < n; ++i) {
      if ((in >> i) & 1ull) continue;
      const int d = manh(pts[best], pts[i]);
      if (d < dist[i]) { dist[i] = d; par[i] = (signed char)best; }
    }
  }
  if (n_edges) *n_edges = ne;
  return total;
}

__device__ void sort_unique(int* v, int& n) {
  for (int i = 1; i < n; ++i) {   // insertion sort (n <= 8)
    const int x = v[i];
    int j = i - 1;
    while (j >= 0 && v[j] > x) { v[j + 1] = v[j]; --j; }
    v[j + 1] = x;
  }
  int m = 0;
  for (int i = 0; i < n; ++i) if (m == 0 || v[m - 1] != v[i]) v[m++] = v[i];
  n = m;
}

// Iterated 1-Steiner (k <= 8 pins): pts = pins then Steiner points; returns their count.
__device__ int one_steiner(const Pt* pins, int k, Pt* pts, unsigned char (*edges)[2], int* n_edges) {
  int xs[8], ys[8], nx = k, ny = k;
  for (int i = 0; i < k; ++i) { xs[i] = pins[i].x; ys[i] = pins[i].y; }
  sort_unique(xs, nx);
  sort_unique(ys, ny);
  int n = k;
  for (int i = 0; i < k; ++i) pts[i] = pins[i];
  int cur = prim(pts, n, 0, true, nullptr, nullptr);
  for (int round = 0; round < 2 * k; ++round) {
    int best = cur, best_c = -1;
    for (int a = 0; a < nx; ++a)
      for (int b = 0; b < ny; ++b) {     // Hanan points in x-major order
        const Pt c{xs[a], ys[b]};
        bool skip = false;
        for (int i = 0; i < n; ++i) if (pts[i].x == c.x && pts[i].y == c.y) { skip = true; break; }   // a pin or already added
        if (skip) continue;
        pts[n] = c;
        const int len = prim(pts, n + 1, 0, true, nullptr, nullptr);
        if (len < best) { best = len; best_c = a * ny + b; }
      }
    if (best_c < 0) break;
    pts[n++] = Pt{xs[best_c / ny], ys[best_c % ny]};
    for (;;) {   // drop Steiner points of degree <= 2
      unsigned char e[kMaxPts][2];
      int ne;
      int deg[kMaxPts];
      prim(pts, n, 0, true, e, &ne);
      for (int i = 0; i < n; ++i) deg[i] = 0;
      for (int q = 0; q < ne; ++q) { deg[e[q][0]]++; deg[e[q][1]]++; }
      int drop = -1;
      for (int j = k; j < n; ++j) if (deg[j] <= 2) { drop = j; break; }
      if (drop < 0) break;
      for (int j = drop; j + 1 < n; ++j) pts[j] = pts[j + 1];
      --n;
    }
    cur = prim(pts, n, 0, true, nullptr, nullptr);
  }
  prim(pts, n, 0, true, edges, n_edges);
  return n;
}

__device__ __forceinline__ short4 canon(Pt a, Pt b) {
  if (a.x > b.x || (a.x == b.x && a.y > b.y)) { const Pt t = a; a = b; b = t; }
  return make_short4((short)a.x, (short)a.y, (short)b.x, (short)b.y);
}
__device__ __forceinline__ bool sub_less(short4 p, short4 q) {
  if (p.x != q.x) return p.x < q.x;
  if (p.y != q.y) return p.y < q.y;
  if (p.z != q.z) return p.z < q.z;
  return p.w < q.w;
}

__device__ __forceinline__ int z_count(int a, int z_cap) {
  if (z_cap < 0 || a < 2) return 0;
  if (z_cap == 0 || a - 1 <= z_cap) return a - 1;
  return z_cap;
}
__device__ __forceinline__ int z_offset(int a, int z_cap, int j) {   // j = 0 .. z_count-1
  if (z_cap == 0 || a - 1 <= z_cap) return j + 1;
  const int den = z_cap + 1;
  return (2 * (j + 1) * a + den) / (2 * den);
}

// C-shape detours (reading Q14b): positions lo-c .. lo-1 then hi+1 .. hi+c, inside [0, n)
__device__ __forceinline__ int c_count(int lo, int hi, int c_cap, int n) {
  return min(c_cap, lo) + min(c_cap, n - 1 - hi);
}
__device__ __forceinline__ int c_position(int lo, int hi, int c_cap, int j) {   // j = 0 .. c_count-1
  const int left = min(c_cap, lo);
  return j < left ? lo - left + j : hi + 1 + (j - left);
}

struct BuildArgs {
  int32_t X, Y, c_cap;
  int64_t n_nets;
  const int64_t* net_pin_off;
  const int2* pin_xy;
  int32_t n_tree_cand, z_cap;
  uint64_t seed;
  short4* subs;        // scratch: kSubPerPin * n_pins
  int64_t* cnt;        // [5][n_nets]: trees, sub-nets, paths, segments, turning points
  int32_t* nsub0;      // sub-nets of tree 0 per net
  // outputs
  int64_t *net_tree_off, *tree_sub_off, *sub_path_off, *path_seg_off, *path_tp_off;
  int4* sub_xy;
  int4* seg;
  int2* tp_xy;
};

__global__ void __launch_bounds__(128) kb_trees(BuildArgs B) {
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (n >= B.n_nets) return;
  const int64_t p0 = B.net_pin_off[n];
  const int k = (int)(B.net_pin_off[n + 1] - p0);
  Pt pins[kMaxPins];
  for (int i = 0; i < k; ++i) { const int2 q = B.pin_xy[p0 + i]; pins[i] = Pt{q.x, q.y}; }
  short4* out = B.subs + kSubPerPin * p0;
  unsigned char e[kMaxPts][2];
  int ne0;
  prim(pins, k, 0, true, e, &ne0);
  for (int q = 0; q < ne0; ++q) out[q] = canon(pins[e[q][0]], pins[e[q][1]]);
  int nsub = ne0, ntree = 1;
  if (B.n_tree_cand >= 2) {
    Pt pts[kMaxPts];
    int ne1;
    if (k <= 8) {
      one_steiner(pins, k, pts, e, &ne1);
    } else {
      for (int i = 0; i < k; ++i) pts[i] = pins[i];
      prim(pts, k, k - 1, false, e, &ne1);
    }
    short4* t1 = out + ne0;
    for (int q = 0; q < ne1; ++q) t1[q] = canon(pts[e[q][0]], pts[e[q][1]]);
    bool same = ne1 == ne0;
    if (same) {   // equal edge sets?  compare sorted copies
      short4 a[kMaxPts], b[kMaxPts];
      for (int q = 0; q < ne0; ++q) { a[q] = out[q]; b[q] = t1[q]; }
      for (int i = 1; i < ne0; ++i) {
        short4 x = a[i]; int j = i - 1;
        while (j >= 0 && sub_less(x, a[j])) { a[j + 1] = a[j]; --j; }
        a[j + 1] = x;
        x = b[i]; j = i - 1;
        while (j >= 0 && sub_less(x, b[j])) { b[j + 1] = b[j]; --j; }
        b[j + 1] = x;
      }
      for (int q = 0; q < ne0 && same; ++q)
        same = a[q].x == b[q].x && a[q].y == b[q].y && a[q].z == b[q].z && a[q].w == b[q].w;
    }
    if (!same) { nsub += ne1; ntree = 2; }
  }
  int64_t np = 0, ns = 0, nt = 0;
  for (int q = 0; q < nsub; ++q) {
    const short4 s = out[q];
    if (s.x == s.z || s.y == s.w) { np += 1; ns += 1; continue; }
    const int nz = z_count(s.z - s.x, B.z_cap) + z_count(abs(s.w - s.y), B.z_cap) +
                   c_count(s.x, s.z, B.c_cap, B.X) + c_count(min(s.y, s.w), max(s.y, s.w), B.c_cap, B.Y);
    np += 2 + nz; ns += 4 + 3 * nz; nt += 2 + 2 * nz;
  }
  B.cnt[n] = ntree;
  B.cnt[B.n_nets + n] = nsub;
  B.cnt[2 * B.n_nets + n] = np;
  B.cnt[3 * B.n_nets + n] = ns;
  B.cnt[4 * B.n_nets + n] = nt;
  B.nsub0[n] = ne0;
}

// exclusive scan, phase 1: per-block sums of kScanBlock elements
__global__ void __launch_bounds__(256) kb_scan_sums(const int64_t* in, int64_t n, int64_t* sums) {
  __shared__ int64_t sh[256];
  const int64_t b0 = (int64_t)blockIdx.x * kScanBlock;
  int64_t s = 0;
  for (int i = threadIdx.x; i < kScanBlock; i += 256) if (b0 + i < n) s += in[b0 + i];
  sh[threadIdx.x] = s;
  __syncthreads();
  for (int o = 128; o > 0; o >>= 1) {
    if (threadIdx.x < o) sh[threadIdx.x] += sh[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) sums[blockIdx.x] = sh[0];
}
// phase 2: exclusive scan of the block sums (one thread; <= a few thousand blocks); total at [nb]
__global__ void kb_scan_sums_scan(int64_t* sums, int64_t nb) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  int64_t run = 0;
  for (int64_t b = 0; b < nb; ++b) { const int64_t v = sums[b]; sums[b] = run; run += v; }
  sums[nb] = run;
}
// phase 3: exclusive scan inside each block, offset by the block's base
__global__ void __launch_bounds__(256) kb_scan_apply(const int64_t* in, int64_t n, const int64_t* sums, int64_t* out) {
  __shared__ int64_t sh[256];
  const int64_t b0 = (int64_t)blockIdx.x * kScanBlock;
  constexpr int per = kScanBlock / 256;
  int64_t v[per], s = 0;
  for (int j = 0; j < per; ++j) {
    const int64_t i = b0 + threadIdx.x * per + j;
    v[j] = i < n ? in[i] : 0;
    s += v[j];
  }
  sh[threadIdx.x] = s;
  __syncthreads();
  for (int o = 1; o < 256; o <<= 1) {   // Hillis-Steele inclusive scan of the thread sums
    const int64_t t = threadIdx.x >= o ? sh[threadIdx.x - o] : 0;
    __syncthreads();
    sh[threadIdx.x] += t;
    __syncthreads();
  }
  int64_t run = sums[blockIdx.x] + sh[threadIdx.x] - s;
  for (int j = 0; j < per; ++j) {
    const int64_t i = b0 + threadIdx.x * per + j;
    if (i < n) out[i] = run;
    run += v[j];
  }
}

__global__ void __launch_bounds__(128) kb_fill(BuildArgs B, const int64_t* off) {
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (n >= B.n_nets) return;
  const int64_t N = B.n_nets;
  int64_t tree = off[n], sub = off[N + n], path = off[2 * N + n], sg = off[3 * N + n], tp = off[4 * N + n];
  const int ntree = (int)B.cnt[n], nsub = (int)B.cnt[N + n], nsub0 = B.nsub0[n];
  const short4* in = B.subs + kSubPerPin * B.net_pin_off[n];
  B.net_tree_off[n] = tree;
  for (int t = 0; t < ntree; ++t) B.tree_sub_off[tree + t] = sub + (t == 0 ? 0 : nsub0);
  for (int q = 0; q < nsub; ++q, ++sub) {
    const short4 s = in[q];
    const int x0 = s.x, y0 = s.y, x1 = s.z, y1 = s.w;
    B.sub_xy[sub] = make_int4(x0, y0, x1, y1);
    B.sub_path_off[sub] = path;
    auto seg = [&](int dir, int line, int a, int b) { B.seg[sg++] = make_int4(dir, line, min(a, b), max(a, b)); };
    auto turn = [&](int x, int y) { B.tp_xy[tp++] = make_int2(x, y); };
    auto done = [&]() { ++path; B.path_seg_off[path] = sg; B.path_tp_off[path] = tp; };
    B.path_seg_off[path] = sg;
    B.path_tp_off[path] = tp;
    if (y0 == y1) { seg(0, y0, x0, x1); done(); continue; }
    if (x0 == x1) { seg(1, x0, y0, y1); done(); continue; }
    seg(0, y0, x0, x1); seg(1, x1, y0, y1); turn(x1, y0); done();   // HV
    seg(1, x0, y0, y1); seg(0, y1, x0, x1); turn(x0, y1); done();   // VH
    const int ax = x1 - x0, nzx = z_count(ax, B.z_cap);
    for (int j = 0; j < nzx; ++j) {                                  // Z-HVH, x_m ascending
      const int xm = x0 + z_offset(ax, B.z_cap, j);
      seg(0, y0, x0, xm); seg(1, xm, y0, y1); seg(0, y1, xm, x1); turn(xm, y0); turn(xm, y1); done();
    }
    const int ylo = min(y0, y1), ay = abs(y1 - y0), nzy = z_count(ay, B.z_cap);
    for (int j = 0; j < nzy; ++j) {                                  // Z-VHV, y_m ascending
      const int ym = ylo + z_offset(ay, B.z_cap, j);
      seg(1, x0, y0, ym); seg(0, ym, x0, x1); seg(1, x1, ym, y1); turn(x0, ym); turn(x1, ym); done();
    }
    const int ncx = c_count(x0, x1, B.c_cap, B.X);
    for (int j = 0; j < ncx; ++j) {                                  // C-HVH, x_m ascending
      const int xm = c_position(x0, x1, B.c_cap, j);
      seg(0, y0, x0, xm); seg(1, xm, y0, y1); seg(0, y1, xm, x1); turn(xm, y0); turn(xm, y1); done();
    }
    const int yhi = max(y0, y1), ncy = c_count(ylo, yhi, B.c_cap, B.Y);
    for (int j = 0; j < ncy; ++j) {                                  // C-VHV, y_m ascending
      const int ym = c_position(ylo, yhi, B.c_cap, j);
      seg(1, x0, y0, ym); seg(0, ym, x0, x1); seg(1, x1, ym, y1); turn(x0, ym); turn(x1, ym); done();
    }
  }
}

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__global__ void __launch_bounds__(256) kb_logits(float* w, int64_t n, uint64_t seed, uint64_t stream) {
  const uint64_t base = mix64(seed + 0x9E3779B97F4A7C15ull * (stream + 1));
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t s = base ^ mix64((uint64_t)i * 0xD1B54A32D192ED03ull + stream);
    s += 0x9E3779B97F4A7C15ull;
    w[i] = (float)((double)(mix64(s) >> 11) * (1.0 / 9007199254740992.0));
  }
}

}  // namespace

struct dgr_built_forest {
  int64_t n_nets = 0, sizes[5] = {0, 0, 0, 0, 0};
  cudaStream_t stream = nullptr;
  int64_t *net_tree_off = nullptr, *tree_sub_off = nullptr, *sub_path_off = nullptr, *path_seg_off = nullptr,
          *path_tp_off = nullptr;
  int4* sub_xy = nullptr;
  int4* seg = nullptr;
  int2* tp_xy = nullptr;
  float *w_tree0 = nullptr, *w_path0 = nullptr;
  void release() {
    void* ptrs[] = {net_tree_off, tree_sub_off, sub_path_off, path_seg_off, path_tp_off, sub_xy, seg, tp_xy, w_tree0, w_path0};
    for (void* p : ptrs) if (p) cudaFreeAsync(p, stream);
  }
};

#define FCUDA(x)                                                                                 \
  do {                                                                                           \
    cudaError_t e_ = (x);                                                                        \
    if (e_ != cudaSuccess) { rc = ffail(DGR_ECUDA, "%s: %s", #x, cudaGetErrorString(e_)); goto done; } \
  } while (0)

extern "C" {

int dgr_build_forest(const dgr_pins_desc* d, void* cuda_stream, dgr_built_forest** out) {
  dgr::clear_error();
  if (!d || !out) return ffail(DGR_EINVAL, "NULL argument");
  *out = nullptr;
  if (d->X < 2 || d->Y < 2 || d->X > 32767 || d->Y > 32767) return ffail(DGR_EINVAL, "grid must be 2..32767 per side");
  if (d->n_nets < 0 || !d->net_pin_off || (d->n_nets > 0 && !d->pin_xy)) return ffail(DGR_EINVAL, "bad pins arrays");
  if (d->n_tree_cand < 1 || d->n_tree_cand > 2) return ffail(DGR_EINVAL, "n_tree_cand must be 1 or 2");
  if (d->c_cap < 0) return ffail(DGR_EINVAL, "c_cap must be >= 0");
  const int64_t N = d->n_nets;
  if (d->net_pin_off[0] != 0) return ffail(DGR_EINVAL, "net_pin_off[0] != 0");
  int64_t bad = -1;
#pragma omp parallel for schedule(dynamic, 4096) reduction(max : bad)
  for (int64_t n = 0; n < N; ++n) {
    const int64_t a = d->net_pin_off[n], b = d->net_pin_off[n + 1];
    bool ok = b - a >= 2 && b - a <= kMaxPins;
    for (int64_t i = a; i < b && ok; ++i) {
      const int x = d->pin_xy[2 * i], y = d->pin_xy[2 * i + 1];
      ok = x >= 0 && x < d->X && y >= 0 && y < d->Y;
      for (int64_t j = a; j < i && ok; ++j) ok = !(d->pin_xy[2 * j] == x && d->pin_xy[2 * j + 1] == y);
    }
    if (!ok) bad = std::max(bad, n);
  }
  if (bad >= 0)
    return ffail(DGR_EINVAL, "net %lld: needs 2..%d distinct pins inside the grid", (long long)bad, kMaxPins);
  const int64_t P = d->net_pin_off[N];
  cudaStream_t s = (cudaStream_t)cuda_stream;
  auto* f = new dgr_built_forest();
  f->n_nets = N;
  f->stream = s;
  int rc = DGR_OK;
  int64_t* pin_off_d = nullptr;
  int2* pins_d = nullptr;
  short4* subs_d = nullptr;
  int64_t *cnt_d = nullptr, *off_d = nullptr, *sums_d = nullptr;
  int32_t* nsub0_d = nullptr;
  int64_t totals[5] = {0, 0, 0, 0, 0};
  const int64_t nblk = (N + kScanBlock - 1) / kScanBlock;
  BuildArgs B{};
  if (N == 0) {
    FCUDA(cudaMallocAsync(&f->net_tree_off, 8, s));
    FCUDA(cudaMallocAsync(&f->tree_sub_off, 8, s));
    FCUDA(cudaMallocAsync(&f->sub_path_off, 8, s));
    FCUDA(cudaMallocAsync(&f->path_seg_off, 8, s));
    FCUDA(cudaMallocAsync(&f->path_tp_off, 8, s));
    FCUDA(cudaMemsetAsync(f->net_tree_off, 0, 8, s));
    FCUDA(cudaMemsetAsync(f->tree_sub_off, 0, 8, s));
    FCUDA(cudaMemsetAsync(f->sub_path_off, 0, 8, s));
    FCUDA(cudaMemsetAsync(f->path_seg_off, 0, 8, s));
    FCUDA(cudaMemsetAsync(f->path_tp_off, 0, 8, s));
    FCUDA(cudaStreamSynchronize(s));
    *out = f;
    return DGR_OK;
  }
  FCUDA(cudaMallocAsync(&pin_off_d, 8 * (N + 1), s));
  FCUDA(cudaMallocAsync(&pins_d, 8 * P, s));
  FCUDA(cudaMallocAsync(&subs_d, 8 * kSubPerPin * P, s));
  FCUDA(cudaMallocAsync(&cnt_d, 8 * 5 * N, s));
  FCUDA(cudaMallocAsync(&off_d, 8 * 5 * N, s));
  FCUDA(cudaMallocAsync(&sums_d, 8 * 5 * (nblk + 1), s));
  FCUDA(cudaMallocAsync(&nsub0_d, 4 * N, s));
  FCUDA(cudaMemcpyAsync(pin_off_d, d->net_pin_off, 8 * (N + 1), cudaMemcpyHostToDevice, s));
  FCUDA(cudaMemcpyAsync(pins_d, d->pin_xy, 8 * P, cudaMemcpyHostToDevice, s));
  B.n_nets = N; B.net_pin_off = pin_off_d; B.pin_xy = pins_d;
  B.n_tree_cand = d->n_tree_cand; B.z_cap = d->z_cap; B.seed = d->seed;
  B.X = d->X; B.Y = d->Y; B.c_cap = d->c_cap;
  B.subs = subs_d; B.cnt = cnt_d; B.nsub0 = nsub0_d;
  kb_trees<<<(unsigned)((N + 127) / 128), 128, 0, s>>>(B);
  for (int a = 0; a < 5; ++a) {
    int64_t* sums = sums_d + a * (nblk + 1);
    kb_scan_sums<<<(unsigned)nblk, 256, 0, s>>>(cnt_d + a * N, N, sums);
    kb_scan_sums_scan<<<1, 32, 0, s>>>(sums, nblk);
    kb_scan_apply<<<(unsigned)nblk, 256, 0, s>>>(cnt_d + a * N, N, sums, off_d + a * N);
    FCUDA(cudaMemcpyAsync(&totals[a], sums + nblk, 8, cudaMemcpyDeviceToHost, s));
  }
  FCUDA(cudaGetLastError());
  FCUDA(cudaStreamSynchronize(s));
  for (int a = 0; a < 5; ++a) f->sizes[a] = totals[a];
  FCUDA(cudaMallocAsync(&f->net_tree_off, 8 * (N + 1), s));
  FCUDA(cudaMallocAsync(&f->tree_sub_off, 8 * (totals[0] + 1), s));
  FCUDA(cudaMallocAsync(&f->sub_path_off, 8 * (totals[1] + 1), s));
  FCUDA(cudaMallocAsync(&f->path_seg_off, 8 * (totals[2] + 1), s));
  FCUDA(cudaMallocAsync(&f->path_tp_off, 8 * (totals[2] + 1), s));
  FCUDA(cudaMallocAsync(&f->sub_xy, 16 * std::max<int64_t>(totals[1], 1), s));
  FCUDA(cudaMallocAsync(&f->seg, 16 * std::max<int64_t>(totals[3], 1), s));
  FCUDA(cudaMallocAsync(&f->tp_xy, 8 * std::max<int64_t>(totals[4], 1), s));
  FCUDA(cudaMallocAsync(&f->w_tree0, 4 * std::max<int64_t>(totals[0], 1), s));
  FCUDA(cudaMallocAsync(&f->w_path0, 4 * std::max<int64_t>(totals[2], 1), s));
  B.net_tree_off = f->net_tree_off; B.tree_sub_off = f->tree_sub_off; B.sub_path_off = f->sub_path_off;
  B.path_seg_off = f->path_seg_off; B.path_tp_off = f->path_tp_off;
  B.sub_xy = f->sub_xy; B.seg = f->seg; B.tp_xy = f->tp_xy;
  kb_fill<<<(unsigned)((N + 127) / 128), 128, 0, s>>>(B, off_d);
  {
    // closing entries of the offset arrays
    const int64_t last[5] = {totals[0], totals[1], totals[2], totals[3], totals[4]};
    FCUDA(cudaMemcpyAsync(f->net_tree_off + N, &last[0], 8, cudaMemcpyHostToDevice, s));
    FCUDA(cudaMemcpyAsync(f->tree_sub_off + totals[0], &last[1], 8, cudaMemcpyHostToDevice, s));
    FCUDA(cudaMemcpyAsync(f->sub_path_off + totals[1], &last[2], 8, cudaMemcpyHostToDevice, s));
    if (totals[0] > 0) {
      kb_logits<<<592, 256, 0, s>>>(f->w_tree0, totals[0], d->seed, 3);
      kb_logits<<<592, 256, 0, s>>>(f->w_path0, totals[2], d->seed, 4);
    }
    FCUDA(cudaGetLastError());
    FCUDA(cudaStreamSynchronize(s));   // `last` lives on this stack frame
  }
done:
  if (pin_off_d) cudaFreeAsync(pin_off_d, s);
  if (pins_d) cudaFreeAsync(pins_d, s);
  if (subs_d) cudaFreeAsync(subs_d, s);
  if (cnt_d) cudaFreeAsync(cnt_d, s);
  if (off_d) cudaFreeAsync(off_d, s);
  if (sums_d) cudaFreeAsync(sums_d, s);
  if (nsub0_d) cudaFreeAsync(nsub0_d, s);
  if (rc != DGR_OK) {
    f->release();
    cudaStreamSynchronize(s);
    delete f;
    return rc;
  }
  *out = f;
  return DGR_OK;
}

int dgr_built_forest_sizes(const dgr_built_forest* f, int64_t sizes[6]) {
  dgr::clear_error();
  if (!f || !sizes) return ffail(DGR_EINVAL, "NULL argument");
  sizes[0] = f->n_nets;
  for (int a = 0; a < 5; ++a) sizes[1 + a] = f->sizes[a];
  return DGR_OK;
}

int dgr_built_forest_download(const dgr_built_forest* f, int64_t* net_tree_off, int64_t* tree_sub_off,
                              int64_t* sub_path_off, int64_t* path_seg_off, int64_t* path_tp_off, int32_t* sub_xy,
                              int32_t* seg, int32_t* tp_xy, float* w_tree0, float* w_path0) {
  dgr::clear_error();
  if (!f) return ffail(DGR_EINVAL, "NULL forest");
  const int64_t N = f->n_nets, T = f->sizes[0], S = f->sizes[1], Pp = f->sizes[2], G = f->sizes[3], TP = f->sizes[4];
  cudaStream_t s = f->stream;
  int rc = DGR_OK;
  auto cp = [&](void* dst, const void* src, size_t bytes) -> cudaError_t {
    if (!bytes || !dst) return cudaSuccess;
    return cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, s);
  };
  FCUDA(cp(net_tree_off, f->net_tree_off, 8 * (N + 1)));
  FCUDA(cp(tree_sub_off, f->tree_sub_off, 8 * (T + 1)));
  FCUDA(cp(sub_path_off, f->sub_path_off, 8 * (S + 1)));
  FCUDA(cp(path_seg_off, f->path_seg_off, 8 * (Pp + 1)));
  FCUDA(cp(path_tp_off, f->path_tp_off, 8 * (Pp + 1)));
  FCUDA(cp(sub_xy, f->sub_xy, 16 * S));
  FCUDA(cp(seg, f->seg, 16 * G));
  FCUDA(cp(tp_xy, f->tp_xy, 8 * TP));
  FCUDA(cp(w_tree0, f->w_tree0, 4 * T));
  FCUDA(cp(w_path0, f->w_path0, 4 * Pp));
  FCUDA(cudaStreamSynchronize(s));
done:
  return rc;
}

int dgr_built_forest_free(dgr_built_forest* f) {
  if (!f) return DGR_OK;
  f->release();
  cudaStreamSynchronize(f->stream);
  delete f;
  return DGR_OK;
}

}  // extern "C"
