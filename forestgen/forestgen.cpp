// forestgen.cpp — deterministic synthetic placement + routing-DAG-forest generator.
//
// Input generator shared by the oracle and the CUDA path (see include/forestgen.h).
// It stands in for the paper's layers L0-L2 (§4.1-4.2):
//   * synthetic placement (nets, pins)          — replaces LEF/DEF input
//   * routing-tree candidates                   — replaces FLUTE / CUGR2 trees:
//       candidate 0 = Prim rectilinear MST, candidate 1 = iterated 1-Steiner on the
//       Hanan grid (k <= 8 pins) else a re-rooted MST; duplicates dropped
//   * tree -> 2-pin sub-nets                    — P:534-536
//   * L-shape path enumeration plus Z-shapes (§3.1) and
//     optional C-shape detours (Q14b, row f4)
//   * capacities per Eq. (1) with a hotspot map
//   * random initial logits w0 ~ U[0,1)
// None of the solver's arithmetic lives here.
#include "forestgen.h"

#include <algorithm>
#include <array>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {

thread_local std::string g_err;

// ---- counter-based RNG (splitmix64 finaliser over (seed, stream, index)) ----
inline uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
struct Rng {
  uint64_t s;
  Rng(uint64_t seed, uint64_t stream, uint64_t idx) {
    s = mix64(seed + 0x9E3779B97F4A7C15ull * (stream + 1)) ^ mix64(idx * 0xD1B54A32D192ED03ull + stream);
  }
  uint64_t next() { s += 0x9E3779B97F4A7C15ull; return mix64(s); }
  double u01() { return (double)(next() >> 11) * 0x1.0p-53; }          // [0,1)
  int uint(int n) { return (int)(u01() * n); }                          // [0,n)
  double normal() {                                                     // Box-Muller
    double u1 = u01(), u2 = u01();
    if (u1 < 1e-300) u1 = 1e-300;
    return std::sqrt(-2.0 * std::log(u1)) * std::cos(6.283185307179586 * u2);
  }
};
enum : uint64_t { ST_NET = 1, ST_HOT = 2, ST_WTREE = 3, ST_WPATH = 4 };

struct Pt { int x, y; };
inline int manh(const Pt& a, const Pt& b) { return std::abs(a.x - b.x) + std::abs(a.y - b.y); }

// Prim MST over pts.  root = start vertex; tie_low: ties to lowest index (else highest).
// Returns edges (parent, child) in insertion order and the total length.
long prim(const std::vector<Pt>& pts, int root, bool tie_low, std::vector<std::pair<int, int>>* edges) {
  const int n = (int)pts.size();
  std::vector<int> dist(n, 1 << 30), par(n, -1);
  std::vector<char> in(n, 0);
  dist[root] = 0;
  long total = 0;
  if (edges) edges->clear();
  for (int it = 0; it < n; ++it) {
    int best = -1;
    for (int i = 0; i < n; ++i) {
      if (in[i]) continue;
      if (best < 0 || dist[i] < dist[best] || (dist[i] == dist[best] && !tie_low)) best = i;
    }
    in[best] = 1;
    total += dist[best];
    if (par[best] >= 0 && edges) edges->push_back({par[best], best});
    for (int i = 0; i < n; ++i) {
      if (in[i]) continue;
      int d = manh(pts[best], pts[i]);
      if (d < dist[i]) { dist[i] = d; par[i] = best; }
    }
  }
  return total;
}

// Iterated 1-Steiner (Kahng-Robins) on the Hanan grid for small pin counts.
void one_steiner(const std::vector<Pt>& pins, std::vector<Pt>* pts_out, std::vector<std::pair<int, int>>* edges) {
  std::vector<int> xs, ys;
  for (auto& p : pins) { xs.push_back(p.x); ys.push_back(p.y); }
  std::sort(xs.begin(), xs.end()); xs.erase(std::unique(xs.begin(), xs.end()), xs.end());
  std::sort(ys.begin(), ys.end()); ys.erase(std::unique(ys.begin(), ys.end()), ys.end());
  std::vector<Pt> cand;
  for (int x : xs)
    for (int y : ys) {
      bool is_pin = false;
      for (auto& p : pins) if (p.x == x && p.y == y) { is_pin = true; break; }
      if (!is_pin) cand.push_back({x, y});
    }
  std::vector<Pt> pts = pins;
  const int k = (int)pins.size();
  long cur = prim(pts, 0, true, nullptr);
  for (int round = 0; round < 2 * k; ++round) {
    long best = cur;
    int best_i = -1;
    for (int i = 0; i < (int)cand.size(); ++i) {
      bool used = false;
      for (int j = k; j < (int)pts.size(); ++j) if (pts[j].x == cand[i].x && pts[j].y == cand[i].y) { used = true; break; }
      if (used) continue;
      pts.push_back(cand[i]);
      long c = prim(pts, 0, true, nullptr);
      pts.pop_back();
      if (c < best) { best = c; best_i = i; }
    }
    if (best_i < 0) break;
    pts.push_back(cand[best_i]);
    // drop Steiner points of degree <= 2 (never increases rectilinear length)
    for (;;) {
      std::vector<std::pair<int, int>> e;
      prim(pts, 0, true, &e);
      std::vector<int> deg(pts.size(), 0);
      for (auto& ed : e) { deg[ed.first]++; deg[ed.second]++; }
      int drop = -1;
      for (int j = k; j < (int)pts.size(); ++j) if (deg[j] <= 2) { drop = j; break; }
      if (drop < 0) break;
      pts.erase(pts.begin() + drop);
    }
    cur = prim(pts, 0, true, nullptr);
  }
  *pts_out = pts;
  prim(pts, 0, true, edges);
}

struct Sub { int x0, y0, x1, y1; };
struct NetOut {
  std::vector<Pt> pins;
  std::vector<int> tree_nsub;          // sub-nets per tree
  std::vector<Sub> subs;
  std::vector<int> sub_npath;          // paths per sub-net
  std::vector<int> path_nseg, path_ntp;
  std::vector<int32_t> seg;            // 4 per segment
  std::vector<int32_t> tp;             // 2 per turning point
};

inline Sub canon(Pt a, Pt b) {
  if (a.x > b.x || (a.x == b.x && a.y > b.y)) std::swap(a, b);
  return {a.x, a.y, b.x, b.y};
}

// interior offsets for Z shapes along a span of length a (a >= 2), capped
void z_offsets(int a, int z_cap, std::vector<int>* off) {
  off->clear();
  if (z_cap < 0 || a < 2) return;
  if (z_cap == 0 || a - 1 <= z_cap) {
    for (int o = 1; o < a; ++o) off->push_back(o);
  } else {
    const int den = z_cap + 1;
    for (int j = 1; j <= z_cap; ++j) off->push_back((2 * j * a + den) / (2 * den));  // floor(j*a/den + 1/2)
  }
}

inline void add_seg(NetOut& o, int dir, int line, int a, int b) {
  o.seg.push_back(dir); o.seg.push_back(line); o.seg.push_back(std::min(a, b)); o.seg.push_back(std::max(a, b));
}
inline void add_tp(NetOut& o, int x, int y) { o.tp.push_back(x); o.tp.push_back(y); }

// C-shape detour positions outside [lo, hi] (reading Q14b): lo-c .. lo-1, then hi+1 .. hi+c, inside [0, n)
void c_positions(int lo, int hi, int c_cap, int n, std::vector<int>* pos) {
  pos->clear();
  for (int d = c_cap; d >= 1; --d) if (lo - d >= 0) pos->push_back(lo - d);
  for (int d = 1; d <= c_cap; ++d) if (hi + d < n) pos->push_back(hi + d);
}

// Monotone staircase corners (row f4', reading Q14c) along a span [lo, hi] of length a >= 3 and
// a cross span of length b >= 2: for k = 1..m_cap, first corner lo + max(1, floor(k a / (2 (m_cap + 1)))),
// second corner half-way from it to hi (strictly inside), cross line lo' + floor(k b / (m_cap + 1))
// clamped strictly inside; duplicates dropped
void stair_corners(int lo, int a, int clo, int b, int m_cap, std::vector<std::array<int, 3>>* out) {
  out->clear();
  if (m_cap <= 0 || a < 3 || b < 2) return;
  for (int k = 1; k <= m_cap; ++k) {
    int p1 = lo + std::max(1, (k * a) / (2 * (m_cap + 1)));
    p1 = std::min(p1, lo + a - 2);
    const int p2 = p1 + std::max(1, (lo + a - p1) / 2);
    int q = clo + (k * b) / (m_cap + 1);
    q = std::min(std::max(q, clo + 1), clo + b - 1);
    const std::array<int, 3> c{p1, std::min(p2, lo + a - 1), q};
    if (std::find(out->begin(), out->end(), c) == out->end()) out->push_back(c);
  }
}

void enumerate_paths(const Sub& s, int z_cap, int c_cap, int m_cap, int X, int Y, NetOut& o) {
  const int x0 = s.x0, y0 = s.y0, x1 = s.x1, y1 = s.y1;
  int np = 0;
  if (y0 == y1) {                       // straight H
    add_seg(o, 0, y0, x0, x1); o.path_nseg.push_back(1); o.path_ntp.push_back(0); np = 1;
  } else if (x0 == x1) {                // straight V
    add_seg(o, 1, x0, y0, y1); o.path_nseg.push_back(1); o.path_ntp.push_back(0); np = 1;
  } else {
    // HV: H on row y0, V on column x1, turn at (x1,y0)
    add_seg(o, 0, y0, x0, x1); add_seg(o, 1, x1, y0, y1); add_tp(o, x1, y0);
    o.path_nseg.push_back(2); o.path_ntp.push_back(1);
    // VH: V on column x0, H on row y1, turn at (x0,y1)
    add_seg(o, 1, x0, y0, y1); add_seg(o, 0, y1, x0, x1); add_tp(o, x0, y1);
    o.path_nseg.push_back(2); o.path_ntp.push_back(1);
    np = 2;
    std::vector<int> off;
    z_offsets(x1 - x0, z_cap, &off);
    for (int d : off) {                 // Z-HVH, x_m ascending
      const int xm = x0 + d;
      add_seg(o, 0, y0, x0, xm); add_seg(o, 1, xm, y0, y1); add_seg(o, 0, y1, xm, x1);
      add_tp(o, xm, y0); add_tp(o, xm, y1);
      o.path_nseg.push_back(3); o.path_ntp.push_back(2); ++np;
    }
    const int ylo = std::min(y0, y1);
    z_offsets(std::abs(y1 - y0), z_cap, &off);
    for (int d : off) {                 // Z-VHV, y_m ascending
      const int ym = ylo + d;
      add_seg(o, 1, x0, y0, ym); add_seg(o, 0, ym, x0, x1); add_seg(o, 1, x1, ym, y1);
      add_tp(o, x0, ym); add_tp(o, x1, ym);
      o.path_nseg.push_back(3); o.path_ntp.push_back(2); ++np;
    }
    c_positions(x0, x1, c_cap, X, &off);
    for (int xm : off) {                // C-HVH, x_m ascending (outside [x0, x1])
      add_seg(o, 0, y0, x0, xm); add_seg(o, 1, xm, y0, y1); add_seg(o, 0, y1, xm, x1);
      add_tp(o, xm, y0); add_tp(o, xm, y1);
      o.path_nseg.push_back(3); o.path_ntp.push_back(2); ++np;
    }
    c_positions(ylo, std::max(y0, y1), c_cap, Y, &off);
    for (int ym : off) {                // C-VHV, y_m ascending (outside [ylo, yhi])
      add_seg(o, 1, x0, y0, ym); add_seg(o, 0, ym, x0, x1); add_seg(o, 1, x1, ym, y1);
      add_tp(o, x0, ym); add_tp(o, x1, ym);
      o.path_nseg.push_back(3); o.path_ntp.push_back(2); ++np;
    }
    // monotone staircases (Q14c): HVHVH turning at x_a, x_b on an intermediate row y_m, then
    // VHVHV turning at y_a, y_b (from y0 towards y1) on an intermediate column x_m
    std::vector<std::array<int, 3>> st;
    const int b = std::abs(y1 - y0), sy = y1 > y0 ? 1 : -1;
    stair_corners(x0, x1 - x0, 0, b, m_cap, &st);
    for (auto& c : st) {
      const int xa = c[0], xb = c[1], ym = y0 + sy * c[2];
      add_seg(o, 0, y0, x0, xa); add_seg(o, 1, xa, y0, ym); add_seg(o, 0, ym, xa, xb);
      add_seg(o, 1, xb, ym, y1); add_seg(o, 0, y1, xb, x1);
      add_tp(o, xa, y0); add_tp(o, xa, ym); add_tp(o, xb, ym); add_tp(o, xb, y1);
      o.path_nseg.push_back(5); o.path_ntp.push_back(4); ++np;
    }
    stair_corners(0, b, x0, x1 - x0, m_cap, &st);
    for (auto& c : st) {
      const int ya = y0 + sy * c[0], yb = y0 + sy * c[1], xm = c[2];
      add_seg(o, 1, x0, y0, ya); add_seg(o, 0, ya, x0, xm); add_seg(o, 1, xm, ya, yb);
      add_seg(o, 0, yb, xm, x1); add_seg(o, 1, x1, yb, y1);
      add_tp(o, x0, ya); add_tp(o, xm, ya); add_tp(o, xm, yb); add_tp(o, x1, yb);
      o.path_nseg.push_back(5); o.path_ntp.push_back(4); ++np;
    }
  }
  o.sub_npath.push_back(np);
}

std::vector<std::pair<Pt, Pt>> canon_edges(const std::vector<Pt>& pts, const std::vector<std::pair<int, int>>& e) {
  std::vector<std::pair<Pt, Pt>> r;
  for (auto& ed : e) {
    Sub s = canon(pts[ed.first], pts[ed.second]);
    r.push_back({{s.x0, s.y0}, {s.x1, s.y1}});
  }
  std::sort(r.begin(), r.end(), [](const std::pair<Pt, Pt>& a, const std::pair<Pt, Pt>& b) {
    if (a.first.x != b.first.x) return a.first.x < b.first.x;
    if (a.first.y != b.first.y) return a.first.y < b.first.y;
    if (a.second.x != b.second.x) return a.second.x < b.second.x;
    return a.second.y < b.second.y;
  });
  return r;
}
bool same_edges(const std::vector<std::pair<Pt, Pt>>& a, const std::vector<std::pair<Pt, Pt>>& b) {
  if (a.size() != b.size()) return false;
  for (size_t i = 0; i < a.size(); ++i)
    if (a[i].first.x != b[i].first.x || a[i].first.y != b[i].first.y ||
        a[i].second.x != b[i].second.x || a[i].second.y != b[i].second.y) return false;
  return true;
}

void build_trees(const forestgen_config& c, NetOut& o) {
  const auto& pins = o.pins;
  const int k = (int)pins.size();
  std::vector<std::pair<int, int>> e0;
  prim(pins, 0, true, &e0);
  std::vector<std::vector<Sub>> trees;
  std::vector<std::vector<std::pair<Pt, Pt>>> keys;
  {
    std::vector<Sub> t;
    for (auto& ed : e0) t.push_back(canon(pins[ed.first], pins[ed.second]));
    trees.push_back(t);
    keys.push_back(canon_edges(pins, e0));
  }
  if (c.n_tree_cand >= 2) {
    std::vector<Pt> pts;
    std::vector<std::pair<int, int>> e1;
    if (k <= 8) {
      one_steiner(pins, &pts, &e1);
    } else {
      pts = pins;
      prim(pts, k - 1, false, &e1);
    }
    auto key = canon_edges(pts, e1);
    if (!same_edges(key, keys[0])) {
      std::vector<Sub> t;
      for (auto& ed : e1) t.push_back(canon(pts[ed.first], pts[ed.second]));
      trees.push_back(t);
    }
  }
  for (auto& t : trees) {
    o.tree_nsub.push_back((int)t.size());
    for (auto& s : t) {
      o.subs.push_back(s);
      enumerate_paths(s, c.z_cap, c.c_cap, c.m_cap, c.X, c.Y, o);
    }
  }
}

inline uint32_t part1by1(uint32_t x) {
  x &= 0xFFFF;
  x = (x | (x << 8)) & 0x00FF00FF;
  x = (x | (x << 4)) & 0x0F0F0F0F;
  x = (x | (x << 2)) & 0x33333333;
  x = (x | (x << 1)) & 0x55555555;
  return x;
}

}  // namespace

struct forestgen_forest {
  forestgen_view v;
  std::vector<int64_t> net_tree_off, tree_sub_off, sub_path_off, path_seg_off, path_tp_off, net_pin_off;
  std::vector<int32_t> seg, tp_xy, sub_xy, pin_xy;
  std::vector<float> cap_h, cap_v, w_tree0, w_path0;
};

extern "C" const char* forestgen_last_error(void) { return g_err.c_str(); }

extern "C" int forestgen_generate(const forestgen_config* cp, forestgen_forest** out) {
  if (!cp || !out) { g_err = "null argument"; return -1; }
  const forestgen_config c = *cp;
  if (c.X < 2 || c.Y < 2 || c.X > 32000 || c.Y > 32000) { g_err = "grid must be 2..32000 per side"; return -1; }
  if (c.n_nets < 0) { g_err = "n_nets < 0"; return -1; }
  if (c.pins_mode == 0 && (c.pins_min < 2 || c.pins_max < c.pins_min)) { g_err = "bad pins range"; return -1; }
  if (c.box_mode == 0 && (c.box_min < 1 || c.box_max < c.box_min)) { g_err = "bad box range"; return -1; }
  if (c.n_tree_cand < 1 || c.n_tree_cand > 2) { g_err = "n_tree_cand must be 1 or 2"; return -1; }
  if (c.c_cap < 0) { g_err = "c_cap < 0"; return -1; }
  if (c.m_cap < 0) { g_err = "m_cap < 0"; return -1; }
  const int X = c.X, Y = c.Y;

  // hotspots (global stream)
  struct Hot { double x, y, s; };
  std::vector<Hot> hot;
  {
    Rng r(c.seed, ST_HOT, 0);
    for (int k = 0; k < c.n_hotspots; ++k) {
      Hot h;
      h.x = r.u01() * X; h.y = r.u01() * Y;
      h.s = X / 40.0 + r.u01() * (X / 10.0 - X / 40.0);
      if (h.s < 0.5) h.s = 0.5;
      hot.push_back(h);
    }
  }

  // ---- nets: placement + trees + paths, one independent RNG stream per net ----
  const int64_t N = c.n_nets;
  std::vector<NetOut> nets(N);
  std::vector<uint32_t> morton(N);
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t g = 0; g < N; ++g) {
    Rng r(c.seed, ST_NET, (uint64_t)g);
    double cx, cy;
    if (!hot.empty() && r.u01() < c.cluster_frac) {
      const Hot& h = hot[r.uint((int)hot.size())];
      cx = h.x + h.s * r.normal();
      cy = h.y + h.s * r.normal();
    } else {
      cx = r.u01() * X;
      cy = r.u01() * Y;
    }
    cx = std::min(std::max(cx, 0.0), X - 1e-9);
    cy = std::min(std::max(cy, 0.0), Y - 1e-9);
    int k;
    if (c.pins_mode == 0) {
      k = c.pins_min + r.uint(c.pins_max - c.pins_min + 1);
    } else {
      int geo = 1;                       // Geom(0.5) on {1,2,...}
      while (geo < 64 && r.u01() >= 0.5) ++geo;
      k = 2 + std::min(geo - 1, 30);
    }
    int b;
    if (c.box_mode == 0) {
      b = c.box_min + r.uint(c.box_max - c.box_min + 1);
    } else {
      double e = -c.box_mu * std::log(1.0 - r.u01());
      b = std::min(X / 2, 2 + (int)std::floor(e));
    }
    b = std::max(1, std::min(b, std::min(X, Y)));
    int bx0 = (int)std::floor(cx - b / 2.0), by0 = (int)std::floor(cy - b / 2.0);
    bx0 = std::min(std::max(bx0, 0), X - b);
    by0 = std::min(std::max(by0, 0), Y - b);
    NetOut& o = nets[g];
    for (int i = 0; i < k; ++i) {
      Pt p{bx0 + r.uint(b), by0 + r.uint(b)};
      bool dup = false;
      for (auto& q : o.pins) if (q.x == p.x && q.y == p.y) { dup = true; break; }
      if (!dup) o.pins.push_back(p);
    }
    if (o.pins.size() >= 2) {
      build_trees(c, o);
      int mnx = X, mxx = -1, mny = Y, mxy = -1;
      for (auto& p : o.pins) { mnx = std::min(mnx, p.x); mxx = std::max(mxx, p.x); mny = std::min(mny, p.y); mxy = std::max(mxy, p.y); }
      morton[g] = part1by1((uint32_t)(mnx + mxx)) | (part1by1((uint32_t)(mny + mxy)) << 1);
    }
  }

  // pin / local-net density (Eq. (1) terms)
  std::vector<int> pin_cnt((size_t)X * Y, 0), local_cnt((size_t)X * Y, 0);
  std::vector<int64_t> routed;
  routed.reserve(N);
  for (int64_t g = 0; g < N; ++g) {
    if (nets[g].pins.size() >= 2) {
      routed.push_back(g);
      for (auto& p : nets[g].pins) pin_cnt[(size_t)p.y * X + p.x]++;
    } else {
      auto& p = nets[g].pins[0];
      local_cnt[(size_t)p.y * X + p.x]++;
    }
  }
  std::stable_sort(routed.begin(), routed.end(), [&](int64_t a, int64_t b) { return morton[a] < morton[b]; });

  auto* f = new forestgen_forest();
  const int64_t NR = (int64_t)routed.size();
  f->net_tree_off.assign(1, 0);
  f->tree_sub_off.assign(1, 0);
  f->sub_path_off.assign(1, 0);
  f->path_seg_off.assign(1, 0);
  f->path_tp_off.assign(1, 0);
  f->net_pin_off.assign(1, 0);
  for (int64_t i = 0; i < NR; ++i) {
    const NetOut& o = nets[routed[i]];
    for (auto& p : o.pins) { f->pin_xy.push_back(p.x); f->pin_xy.push_back(p.y); }
    f->net_pin_off.push_back((int64_t)f->pin_xy.size() / 2);
    for (int nt : o.tree_nsub) f->tree_sub_off.push_back(f->tree_sub_off.back() + nt);
    f->net_tree_off.push_back((int64_t)f->tree_sub_off.size() - 1);
    for (size_t s = 0; s < o.subs.size(); ++s) {
      const Sub& sb = o.subs[s];
      f->sub_xy.push_back(sb.x0); f->sub_xy.push_back(sb.y0); f->sub_xy.push_back(sb.x1); f->sub_xy.push_back(sb.y1);
      f->sub_path_off.push_back(f->sub_path_off.back() + o.sub_npath[s]);
    }
    for (size_t p = 0; p < o.path_nseg.size(); ++p) {
      f->path_seg_off.push_back(f->path_seg_off.back() + o.path_nseg[p]);
      f->path_tp_off.push_back(f->path_tp_off.back() + o.path_ntp[p]);
    }
    f->seg.insert(f->seg.end(), o.seg.begin(), o.seg.end());
    f->tp_xy.insert(f->tp_xy.end(), o.tp.begin(), o.tp.end());
  }
  const int64_t NT = (int64_t)f->tree_sub_off.size() - 1;
  const int64_t NP = (int64_t)f->path_seg_off.size() - 1;

  // capacities, Eq. (1): cap_e = T*h(e) - beta_pin*(pins(a)+pins(b))/2 - (local(a)+local(b))/2,
  // rounded to multiples of 1/4
  std::vector<double> hh((size_t)(2 * X) * (2 * Y), 0.0);   // hotspot sum sampled on the half-cell lattice
  for (auto& h : hot) {
    const double rad = 6.0 * h.s;
    int ax0 = std::max(0, (int)std::floor(2 * (h.x - rad))), ax1 = std::min(2 * X - 1, (int)std::ceil(2 * (h.x + rad)));
    int ay0 = std::max(0, (int)std::floor(2 * (h.y - rad))), ay1 = std::min(2 * Y - 1, (int)std::ceil(2 * (h.y + rad)));
    for (int j = ay0; j <= ay1; ++j)
      for (int i = ax0; i <= ax1; ++i) {
        const double px = 0.5 * i, py = 0.5 * j, dx = px - h.x, dy = py - h.y;
        hh[(size_t)j * (2 * X) + i] += std::exp(-(dx * dx + dy * dy) / (2 * h.s * h.s));
      }
  }
  auto hval = [&](int i2, int j2) {   // h at continuous point (i2/2, j2/2)
    double v = 1.0 - 0.7 * hh[(size_t)j2 * (2 * X) + i2];
    return v < 0.1 ? 0.1 : v;
  };
  auto q4 = [](double v) { return (float)(std::floor(v * 4.0 + 0.5) / 4.0); };
  f->cap_h.assign((size_t)X * Y, 0.f);
  f->cap_v.assign((size_t)X * Y, 0.f);
  for (int y = 0; y < Y; ++y)
    for (int x = 0; x < X; ++x) {
      const size_t a = (size_t)y * X + x;
      if (x + 1 < X) {
        const size_t b = a + 1;
        double v = c.track * hval(2 * x + 2 < 2 * X ? 2 * x + 2 : 2 * X - 1, 2 * y + 1) -
                   c.beta_pin * (pin_cnt[a] + pin_cnt[b]) / 2.0 - c.local_weight * (local_cnt[a] + local_cnt[b]) / 2.0;
        f->cap_h[a] = q4(v);
      }
      if (y + 1 < Y) {
        const size_t b = a + X;
        double v = c.track * hval(2 * x + 1, 2 * y + 2 < 2 * Y ? 2 * y + 2 : 2 * Y - 1) -
                   c.beta_pin * (pin_cnt[a] + pin_cnt[b]) / 2.0 - c.local_weight * (local_cnt[a] + local_cnt[b]) / 2.0;
        f->cap_v[a] = q4(v);
      }
    }

  // random initial logits, U[0,1)
  f->w_tree0.resize(NT);
  f->w_path0.resize(NP);
  for (int64_t j = 0; j < NT; ++j) { Rng r(c.seed, ST_WTREE, (uint64_t)j); f->w_tree0[j] = (float)r.u01(); }
  for (int64_t i = 0; i < NP; ++i) { Rng r(c.seed, ST_WPATH, (uint64_t)i); f->w_path0[i] = (float)r.u01(); }

  forestgen_view& v = f->v;
  v.X = X; v.Y = Y;
  v.n_nets = NR; v.n_trees = NT; v.n_subnets = (int64_t)f->sub_path_off.size() - 1; v.n_paths = NP;
  v.n_segs = (int64_t)f->seg.size() / 4; v.n_tps = (int64_t)f->tp_xy.size() / 2;
  v.n_local_nets = N - NR; v.n_pins = (int64_t)f->pin_xy.size() / 2;
  v.net_tree_off = f->net_tree_off.data(); v.tree_sub_off = f->tree_sub_off.data();
  v.sub_path_off = f->sub_path_off.data(); v.path_seg_off = f->path_seg_off.data();
  v.path_tp_off = f->path_tp_off.data();
  v.seg = f->seg.data(); v.tp_xy = f->tp_xy.data(); v.sub_xy = f->sub_xy.data();
  v.cap_h = f->cap_h.data(); v.cap_v = f->cap_v.data();
  v.w_tree0 = f->w_tree0.data(); v.w_path0 = f->w_path0.data();
  v.net_pin_off = f->net_pin_off.data(); v.pin_xy = f->pin_xy.data();
  *out = f;
  return 0;
}

extern "C" void forestgen_get_view(const forestgen_forest* f, forestgen_view* v) { *v = f->v; }
extern "C" void forestgen_free(forestgen_forest* f) { delete f; }
