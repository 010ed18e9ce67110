/* forest_oracle.c — PARITY ORACLE for row f1 (routing-DAG-forest construction).  TEST
 * INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it; the product path never links or calls it.
 *
 * A plain, single-threaded C statement of §4.2 of the paper under the
 * readings of DESIGN.md §3:
 *   routing-tree candidates per net (the paper uses FLUTE and CUGR2's variant, which
 *     are not available — reading Q17): candidate 0 = Prim's rectilinear MST rooted at pin 0,
 *     ties to the lowest index; candidate 1 = iterated 1-Steiner on the Hanan grid (Kahng-Robins)
 *     for nets of <= 8 pins, else Prim rooted at the last pin with ties to the highest index;
 *     candidate 1 is dropped when its edge set equals candidate 0's;
 *   2-pin sub-nets = the tree edges, in the order Prim adds them, endpoints canonical
 *     (x0 <= x1; y0 < y1 if x0 == x1);
 *   path candidates per sub-net (§3.1, reading Q14): the straight path if
 *     aligned, else HV, VH, Z-HVH (x_m ascending), Z-VHV (y_m ascending); at most z_cap Z per
 *     direction at offsets floor(j a/(z_cap+1) + 1/2) (z_cap 0 = all, -1 = none); then the
 *     C-shape detours of reading Q14b (row f4): C-HVH at x_m = x0-c_cap .. x0-1, x1+1 .. x1+c_cap,
 *     C-VHV at y_m = ylo-c_cap .. ylo-1, yhi+1 .. yhi+c_cap, those inside the grid;
 *   initial logits w0 ~ U[0,1) (reading Q8): a splitmix64-finalised counter hash of
 *     (seed, stream 3 trees / 4 paths, global index), 53 random bits.
 * No blocking, no parallelism, no incremental MST: every candidate evaluation re-runs Prim.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ODGR_API __attribute__((visibility("default")))

typedef struct { int x, y; } opt_t;

static int manh(opt_t a, opt_t b) { return abs(a.x - b.x) + abs(a.y - b.y); }

/* Prim over pts[0..n), started at `root`; tie_low: among equal keys the lowest index, else the
 * highest.  Writes the edges (parent, child) in the order vertices join; returns the length. */
static long prim(const opt_t* pts, int n, int root, int tie_low, int (*edges)[2], int* n_edges) {
  int dist[64], par[64], in[64];
  for (int i = 0; i < n; ++i) { dist[i] = 1 << 30; par[i] = -1; in[i] = 0; }
  dist[root] = 0;
  long total = 0;
  int ne = 0;
  for (int it = 0; it < n; ++it) {
    int best = -1;
    for (int i = 0; i < n; ++i) {
      if (in[i]) continue;
      if (best < 0 || dist[i] < dist[best] || (dist[i] == dist[best] && !tie_low)) best = i;
    }
    in[best] = 1;
    total += dist[best];
    if (par[best] >= 0) {
      if (edges) { edges[ne][0] = par[best]; edges[ne][1] = best; }
      ++ne;
    }
    for (int i = 0; i < n; ++i) {
      if (in[i]) continue;
      int d = manh(pts[best], pts[i]);
      if (d < dist[i]) { dist[i] = d; par[i] = best; }
    }
  }
  if (n_edges) *n_edges = ne;
  return total;
}

static int cmp_int(const void* a, const void* b) { return (*(const int*)a > *(const int*)b) - (*(const int*)a < *(const int*)b); }

/* Iterated 1-Steiner on the Hanan grid of the k pins: each round adds the Hanan point (x-major
 * order, not a pin, not already added) that lowers the MST length the most (strictly), then
 * removes added points of MST degree <= 2 (the first one, repeatedly); at most 2k rounds.
 * pts receives pins then Steiner points; returns their count. */
static int one_steiner(const opt_t* pins, int k, opt_t* pts, int (*edges)[2], int* n_edges) {
  int xs[32], ys[32], nx = 0, ny = 0;
  for (int i = 0; i < k; ++i) { xs[i] = pins[i].x; ys[i] = pins[i].y; }
  qsort(xs, k, sizeof(int), cmp_int);
  qsort(ys, k, sizeof(int), cmp_int);
  for (int i = 0; i < k; ++i) if (nx == 0 || xs[nx - 1] != xs[i]) xs[nx++] = xs[i];
  for (int i = 0; i < k; ++i) if (ny == 0 || ys[ny - 1] != ys[i]) ys[ny++] = ys[i];
  opt_t cand[1024];
  int nc = 0;
  for (int a = 0; a < nx; ++a)
    for (int b = 0; b < ny; ++b) {
      int is_pin = 0;
      for (int i = 0; i < k; ++i) if (pins[i].x == xs[a] && pins[i].y == ys[b]) { is_pin = 1; break; }
      if (!is_pin) { cand[nc].x = xs[a]; cand[nc].y = ys[b]; ++nc; }
    }
  int n = k;
  for (int i = 0; i < k; ++i) pts[i] = pins[i];
  long cur = prim(pts, n, 0, 1, NULL, NULL);
  for (int round = 0; round < 2 * k; ++round) {
    long best = cur;
    int best_i = -1;
    for (int i = 0; i < nc; ++i) {
      int used = 0;
      for (int j = k; j < n; ++j) if (pts[j].x == cand[i].x && pts[j].y == cand[i].y) { used = 1; break; }
      if (used) continue;
      pts[n] = cand[i];
      long c = prim(pts, n + 1, 0, 1, NULL, NULL);
      if (c < best) { best = c; best_i = i; }
    }
    if (best_i < 0) break;
    pts[n++] = cand[best_i];
    for (;;) {   /* drop Steiner points of degree <= 2 (they never shorten a rectilinear tree) */
      int e[64][2], ne, deg[64] = {0};
      prim(pts, n, 0, 1, e, &ne);
      for (int q = 0; q < ne; ++q) { deg[e[q][0]]++; deg[e[q][1]]++; }
      int drop = -1;
      for (int j = k; j < n; ++j) if (deg[j] <= 2) { drop = j; break; }
      if (drop < 0) break;
      for (int j = drop; j + 1 < n; ++j) pts[j] = pts[j + 1];
      --n;
    }
    cur = prim(pts, n, 0, 1, NULL, NULL);
  }
  prim(pts, n, 0, 1, edges, n_edges);
  return n;
}

/* canonical endpoints of a sub-net: x0 <= x1, and y0 < y1 when x0 == x1 */
static void canon(opt_t a, opt_t b, int out[4]) {
  if (a.x > b.x || (a.x == b.x && a.y > b.y)) { opt_t t = a; a = b; b = t; }
  out[0] = a.x; out[1] = a.y; out[2] = b.x; out[3] = b.y;
}
static int cmp_sub(const void* a, const void* b) {
  const int* p = (const int*)a; const int* q = (const int*)b;
  for (int i = 0; i < 4; ++i) if (p[i] != q[i]) return p[i] < q[i] ? -1 : 1;
  return 0;
}

/* ---- growable arrays ---- */
typedef struct { void* p; size_t n, cap, esz; } ovec;
static void ov_init(ovec* v, size_t esz) { v->p = NULL; v->n = 0; v->cap = 0; v->esz = esz; }
static void* ov_push(ovec* v) {
  if (v->n == v->cap) { v->cap = v->cap ? 2 * v->cap : 1024; v->p = realloc(v->p, v->cap * v->esz); }
  return (char*)v->p + (v->n++) * v->esz;
}
static void ov_i64(ovec* v, int64_t x) { *(int64_t*)ov_push(v) = x; }
static void ov_i32(ovec* v, int32_t x) { *(int32_t*)ov_push(v) = x; }

typedef struct {
  ovec net_tree_off, tree_sub_off, sub_path_off, path_seg_off, path_tp_off;   /* int64 */
  ovec sub_xy, seg, tp_xy;                                                    /* int32 */
  float *w_tree0, *w_path0;
} odgr_forest;

/* Z offsets along a span of a >= 2 cells (reading Q14) */
static int z_offsets(int a, int z_cap, int* off) {
  int n = 0;
  if (z_cap < 0 || a < 2) return 0;
  if (z_cap == 0 || a - 1 <= z_cap) {
    for (int o = 1; o < a; ++o) off[n++] = o;
  } else {
    int den = z_cap + 1;
    for (int j = 1; j <= z_cap; ++j) off[n++] = (2 * j * a + den) / (2 * den);
  }
  return n;
}

static void add_seg(odgr_forest* f, int dir, int line, int a, int b) {
  ov_i32(&f->seg, dir); ov_i32(&f->seg, line); ov_i32(&f->seg, a < b ? a : b); ov_i32(&f->seg, a < b ? b : a);
}
static void add_tp(odgr_forest* f, int x, int y) { ov_i32(&f->tp_xy, x); ov_i32(&f->tp_xy, y); }
static void end_path(odgr_forest* f) {
  ov_i64(&f->path_seg_off, (int64_t)(f->seg.n / 4));
  ov_i64(&f->path_tp_off, (int64_t)(f->tp_xy.n / 2));
}

/* the path candidates of one canonical sub-net (x0,y0)-(x1,y1) */
static void enumerate(odgr_forest* f, const int s[4], int z_cap, int c_cap, int X, int Y) {
  const int x0 = s[0], y0 = s[1], x1 = s[2], y1 = s[3];
  const int ylo = y0 < y1 ? y0 : y1, yhi = y0 < y1 ? y1 : y0;
  if (y0 == y1) { add_seg(f, 0, y0, x0, x1); end_path(f); }
  else if (x0 == x1) { add_seg(f, 1, x0, y0, y1); end_path(f); }
  else {
    add_seg(f, 0, y0, x0, x1); add_seg(f, 1, x1, y0, y1); add_tp(f, x1, y0); end_path(f);   /* HV */
    add_seg(f, 1, x0, y0, y1); add_seg(f, 0, y1, x0, x1); add_tp(f, x0, y1); end_path(f);   /* VH */
    static int off[32768];   /* grid sides <= 32767 */
    int n = z_offsets(x1 - x0, z_cap, off);
    for (int q = 0; q < n; ++q) {                                                              /* Z-HVH */
      int xm = x0 + off[q];
      add_seg(f, 0, y0, x0, xm); add_seg(f, 1, xm, y0, y1); add_seg(f, 0, y1, xm, x1);
      add_tp(f, xm, y0); add_tp(f, xm, y1); end_path(f);
    }
    n = z_offsets(yhi - ylo, z_cap, off);
    for (int q = 0; q < n; ++q) {                                                              /* Z-VHV */
      int ym = ylo + off[q];
      add_seg(f, 1, x0, y0, ym); add_seg(f, 0, ym, x0, x1); add_seg(f, 1, x1, ym, y1);
      add_tp(f, x0, ym); add_tp(f, x1, ym); end_path(f);
    }
    for (int side = 0; side < 2; ++side)                                                       /* C-HVH */
      for (int q = 0; q < c_cap; ++q) {
        const int xm = side == 0 ? x0 - (c_cap - q) : x1 + 1 + q;
        if (xm < 0 || xm >= X) continue;
        add_seg(f, 0, y0, x0, xm); add_seg(f, 1, xm, y0, y1); add_seg(f, 0, y1, xm, x1);
        add_tp(f, xm, y0); add_tp(f, xm, y1); end_path(f);
      }
    for (int side = 0; side < 2; ++side)                                                       /* C-VHV */
      for (int q = 0; q < c_cap; ++q) {
        const int ym = side == 0 ? ylo - (c_cap - q) : yhi + 1 + q;
        if (ym < 0 || ym >= Y) continue;
        add_seg(f, 1, x0, y0, ym); add_seg(f, 0, ym, x0, x1); add_seg(f, 1, x1, ym, y1);
        add_tp(f, x0, ym); add_tp(f, x1, ym); end_path(f);
      }
  }
  ov_i64(&f->sub_path_off, (int64_t)(f->path_seg_off.n - 1));
}

/* U[0,1) of (seed, stream, index): splitmix64 finaliser over a counter (reading Q8) */
static uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static double u01(uint64_t seed, uint64_t stream, uint64_t idx) {
  uint64_t s = mix64(seed + 0x9E3779B97F4A7C15ull * (stream + 1)) ^ mix64(idx * 0xD1B54A32D192ED03ull + stream);
  s += 0x9E3779B97F4A7C15ull;
  return (double)(mix64(s) >> 11) * (1.0 / 9007199254740992.0);
}

ODGR_API odgr_forest* odgr_build_forest(int32_t X, int32_t Y, int64_t n_nets, const int64_t* net_pin_off,
                                        const int32_t* pin_xy, int32_t n_tree_cand, int32_t z_cap, int32_t c_cap,
                                        uint64_t seed) {
  odgr_forest* f = (odgr_forest*)calloc(1, sizeof(odgr_forest));
  ov_init(&f->net_tree_off, 8); ov_init(&f->tree_sub_off, 8); ov_init(&f->sub_path_off, 8);
  ov_init(&f->path_seg_off, 8); ov_init(&f->path_tp_off, 8);
  ov_init(&f->sub_xy, 4); ov_init(&f->seg, 4); ov_init(&f->tp_xy, 4);
  ov_i64(&f->net_tree_off, 0); ov_i64(&f->tree_sub_off, 0); ov_i64(&f->sub_path_off, 0);
  ov_i64(&f->path_seg_off, 0); ov_i64(&f->path_tp_off, 0);
  for (int64_t n = 0; n < n_nets; ++n) {
    const int k = (int)(net_pin_off[n + 1] - net_pin_off[n]);
    opt_t pins[32];
    for (int i = 0; i < k; ++i) { pins[i].x = pin_xy[2 * (net_pin_off[n] + i)]; pins[i].y = pin_xy[2 * (net_pin_off[n] + i) + 1]; }
    /* candidate 0: MST from pin 0 */
    int e0[64][2], ne0;
    prim(pins, k, 0, 1, e0, &ne0);
    int t0[64][4], t1[64][4], nt1 = 0, have1 = 0;
    for (int q = 0; q < ne0; ++q) canon(pins[e0[q][0]], pins[e0[q][1]], t0[q]);
    if (n_tree_cand >= 2) {
      opt_t pts[64];
      int e1[64][2], ne1;
      if (k <= 8) {
        one_steiner(pins, k, pts, e1, &ne1);
      } else {
        for (int i = 0; i < k; ++i) pts[i] = pins[i];
        prim(pts, k, k - 1, 0, e1, &ne1);
      }
      for (int q = 0; q < ne1; ++q) canon(pts[e1[q][0]], pts[e1[q][1]], t1[q]);
      nt1 = ne1;
      /* drop a duplicate of candidate 0 (same edge set) */
      int same = ne1 == ne0;
      if (same) {
        int a[64][4], b[64][4];
        memcpy(a, t0, sizeof(int) * 4 * ne0);
        memcpy(b, t1, sizeof(int) * 4 * ne1);
        qsort(a, ne0, sizeof(a[0]), cmp_sub);
        qsort(b, ne1, sizeof(b[0]), cmp_sub);
        same = memcmp(a, b, sizeof(int) * 4 * ne0) == 0;
      }
      have1 = !same;
    }
    for (int t = 0; t < 1 + have1; ++t) {
      int (*tr)[4] = t == 0 ? t0 : t1;
      int ne = t == 0 ? ne0 : nt1;
      for (int q = 0; q < ne; ++q) {
        for (int c = 0; c < 4; ++c) ov_i32(&f->sub_xy, tr[q][c]);
        enumerate(f, tr[q], z_cap, c_cap, X, Y);
      }
      ov_i64(&f->tree_sub_off, (int64_t)(f->sub_xy.n / 4));
    }
    ov_i64(&f->net_tree_off, (int64_t)(f->tree_sub_off.n - 1));
  }
  const int64_t nt = (int64_t)f->tree_sub_off.n - 1, np = (int64_t)f->path_seg_off.n - 1;
  f->w_tree0 = (float*)malloc(sizeof(float) * (nt + 1));
  f->w_path0 = (float*)malloc(sizeof(float) * (np + 1));
  for (int64_t j = 0; j < nt; ++j) f->w_tree0[j] = (float)u01(seed, 3, (uint64_t)j);
  for (int64_t i = 0; i < np; ++i) f->w_path0[i] = (float)u01(seed, 4, (uint64_t)i);
  return f;
}

/* trees, sub-nets, paths, segments, turning points */
ODGR_API void odgr_forest_sizes(const odgr_forest* f, int64_t out[5]) {
  out[0] = (int64_t)f->tree_sub_off.n - 1; out[1] = (int64_t)f->sub_path_off.n - 1;
  out[2] = (int64_t)f->path_seg_off.n - 1; out[3] = (int64_t)f->seg.n / 4; out[4] = (int64_t)f->tp_xy.n / 2;
}

ODGR_API void odgr_forest_copy(const odgr_forest* f, int64_t* net_tree_off, int64_t* tree_sub_off,
                               int64_t* sub_path_off, int64_t* path_seg_off, int64_t* path_tp_off,
                               int32_t* sub_xy, int32_t* seg, int32_t* tp_xy, float* w_tree0, float* w_path0) {
  memcpy(net_tree_off, f->net_tree_off.p, 8 * f->net_tree_off.n);
  memcpy(tree_sub_off, f->tree_sub_off.p, 8 * f->tree_sub_off.n);
  memcpy(sub_path_off, f->sub_path_off.p, 8 * f->sub_path_off.n);
  memcpy(path_seg_off, f->path_seg_off.p, 8 * f->path_seg_off.n);
  memcpy(path_tp_off, f->path_tp_off.p, 8 * f->path_tp_off.n);
  if (f->sub_xy.n) memcpy(sub_xy, f->sub_xy.p, 4 * f->sub_xy.n);
  if (f->seg.n) memcpy(seg, f->seg.p, 4 * f->seg.n);
  if (f->tp_xy.n) memcpy(tp_xy, f->tp_xy.p, 4 * f->tp_xy.n);
  memcpy(w_tree0, f->w_tree0, sizeof(float) * (f->tree_sub_off.n - 1));
  memcpy(w_path0, f->w_path0, sizeof(float) * (f->path_seg_off.n - 1));
}

ODGR_API void odgr_forest_free(odgr_forest* f) {
  if (!f) return;
  free(f->net_tree_off.p); free(f->tree_sub_off.p); free(f->sub_path_off.p); free(f->path_seg_off.p);
  free(f->path_tp_off.p); free(f->sub_xy.p); free(f->seg.p); free(f->tp_xy.p);
  free(f->w_tree0); free(f->w_path0);
  free(f);
}
