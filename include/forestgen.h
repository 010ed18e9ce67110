/* forestgen.h — deterministic synthetic placement + DAG-forest generator (C ABI).
 *
 * This is the shared INPUT generator: both the oracle (oracle/) and the CUDA
 * path (libdgr) consume what it emits.  It holds none of the solver's
 * arithmetic (no softmax, demand, loss, gradient, Adam or induction); it only
 * synthesises what the paper's layers L0-L2 would produce (§4.2,
 * lines 524-539): nets, routing-tree candidates, their 2-pin
 * sub-nets, the L- and Z-shape path candidates of every sub-net
 * (P:536-537 and §3.1), G-cell edge capacities per Eq. (1)
 * and random initial logits w0.
 *
 * Determinism: every random draw is a counter-based hash of (seed, net id,
 * draw index), so the output is identical for any thread count.
 *
 * Geometry conventions (shared with include/dgr.h):
 *   G-cell grid X x Y.  H edge (x,y)-(x+1,y) for x in [0,X-2]; V edge
 *   (x,y)-(x,y+1) for y in [0,Y-2].  Grids are row-major [Y][X]; the unused
 *   last column (H) / last row (V) is padding and holds 0.
 *   Segment = {dir (0=H,1=V), line (y for H, x for V), lo, hi}: the edges
 *   [lo,hi) of that line.  Turning point = {x,y}.
 *   Sub-net endpoints are emitted canonically: x0 <= x1 and, if x0 == x1,
 *   y0 < y1.  Path candidate order per sub-net: the straight path if the
 *   sub-net is aligned, else [HV, VH, Z-HVH by x_m ascending, Z-VHV by y_m
 *   ascending, C-HVH by x_m ascending, C-VHV by y_m ascending, staircases HVHVH then VHVHV]
 *   (
 *   C-shapes, Q14b: x_m in [x0-c_cap, x0-1] then [x1+1, x1+c_cap], y_m in
 *   [ylo-c_cap, ylo-1] then [yhi+1, yhi+c_cap], inside the grid).
 *   Nets are emitted in Morton order of their pin bounding-box centre.
 */
#ifndef FORESTGEN_H
#define FORESTGEN_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  int32_t X, Y;            /* G-cell grid */
  int64_t n_nets;          /* nets to draw (single-cell nets become local nets) */
  int32_t pins_mode;       /* 0: k ~ U{pins_min..pins_max}; 1: k = 2 + min(Geom(0.5)-1, 30) */
  int32_t pins_min, pins_max;
  int32_t box_mode;        /* 0: side b ~ U{box_min..box_max}; 1: b = min(X/2, 2 + floor(Exp(box_mu))) */
  int32_t box_min, box_max;
  double  box_mu;
  double  cluster_frac;    /* fraction of nets whose centre is drawn around a hotspot */
  int32_t n_hotspots;      /* 0 = uniform capacity map */
  double  track;           /* T: tracks per edge before the hotspot map */
  double  beta_pin;        /* pin-density weight of Eq. (1) */
  int32_t n_tree_cand;     /* 1 or 2 routing-tree candidates per net */
  int32_t z_cap;           /* -1: L only; 0: all Z; >0: at most z_cap Z per direction */
  uint64_t seed;
  double  local_weight;    /* weight of the local-net term of Eq. (1) (1 = as written; 0 for Table 1's uniform cap) */
  int32_t c_cap;           /* C-shape detours per side of a non-aligned sub-net (0 = none; reading Q14b) */
  int32_t m_cap;           /* monotone staircases per orientation (0 = none; row f4, reading Q14c): HVHVH
                              and VHVHV paths with four turning points, after the C-shapes */
} forestgen_config;

typedef struct forestgen_forest forestgen_forest;

typedef struct {
  int32_t X, Y;
  int64_t n_nets, n_trees, n_subnets, n_paths, n_segs, n_tps, n_local_nets, n_pins;
  const int64_t *net_tree_off, *tree_sub_off, *sub_path_off, *path_seg_off, *path_tp_off;
  const int32_t *seg;      /* n_segs x 4 */
  const int32_t *tp_xy;    /* n_tps x 2 */
  const int32_t *sub_xy;   /* n_subnets x 4 */
  const float   *cap_h, *cap_v;      /* [Y][X] */
  const float   *w_tree0, *w_path0;  /* U[0,1) initial logits */
  const int64_t *net_pin_off;        /* n_nets+1 */
  const int32_t *pin_xy;             /* n_pins x 2 (deduplicated pins of routed nets) */
} forestgen_view;

/* 0 on success, <0 on invalid config.  *out owns all arrays. */
int  forestgen_generate(const forestgen_config* cfg, forestgen_forest** out);
void forestgen_get_view(const forestgen_forest* f, forestgen_view* v);
void forestgen_free(forestgen_forest* f);
const char* forestgen_last_error(void);

#ifdef __cplusplus
}
#endif
#endif
