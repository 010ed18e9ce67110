/* dgr_oracle.c — the PARITY ORACLE for the DGR solver iteration.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  The product path (paper_conf_dac_0159layhrr24_b200)
 * never links, imports or calls it, and shares no code, header, table or helper
 * with it.
 *
 * A plain, deliberately naive, single-threaded fp64 CPU implementation of what the
 * DGR differentiable solver computes, written from the paper (/root/reference/PAPER.md,
 * "P:NNN" = line NNN) in the paper's order and notation:
 *
 *   Gumbel noise g ~ Gumbel(0,1)                 §4.4, P:817-832 (reading Q7: Philox4x32-10;
 *                                                  a lone straight candidate draws none, the
 *                                                  others are numbered in forest order)
 *   p_i = softmax_{subnet(i)}((w_i+g_i)/t)        §4.4, P:820-826 (reading Q1: group = sub-net)
 *   q_j = softmax_{net(j)}((w_j+g_j)/t)           §4.4
 *   d_e = sum_{i in P_e} q p + beta sum_{k in P_v} q p     Eq. (10), P:556-564 (reading Q3)
 *   overflow_cost = sum_e f(cap_e - d_e)           Eq. (9),  P:550-554 (readings Q2, Q10)
 *   wirelength_cost = sum_i q p WL_i               Eq. (11), P:566-570 (reading Q5)
 *   via_cost = sqrt(L) sum_i q p TP_i              Eq. (12), P:572-578 (readings Q4, Q22)
 *   cost = 500 overflow + 4 via + 0.5 WL
 *   gradient of the cost w.r.t. w                  P:841-847 (autograd in the paper; here the
 *                                                  chain rule written out, pinned by finite
 *                                                  differences and torch autograd in tests/)
 *   Adam, lr 0.3, torch defaults                   P:913-914 (reading Q9)
 *   annealing t_k = 0.9^floor(k/100)               P:915-917 (host schedule, reading Q6)
 *   argmax tree, top-p paths                       §4.5, P:849-861 (readings Q12, Q13, Q23)
 *
 * Demand is rasterised edge by edge; no difference arrays, no prefix sums, no
 * fixed point: those are implementation devices of the CUDA path, not the method.
 * Readings (Q-numbers) are listed in DESIGN.md §3.
 */
#include <stdint.h>
#include <tgmath.h>   /* type-generic exp/log/sqrt/pow/fabs: follow `real` below */
#include <stdlib.h>
#include <string.h>

#define ODGR_API __attribute__((visibility("default")))

/* The oracle computes in `real` = double (fp64, the parity reference).  The same source built with
 * -DODGR_REAL=float is used ONLY as a conditioning probe: it shows which outputs fp32 arithmetic
 * cannot determine to the parity tolerance (reading Q21b).  The ABI stays double. */
#ifndef ODGR_REAL
#define ODGR_REAL double
#endif
typedef ODGR_REAL real;
#define R(x) ((real)(x))

/* ------------------------------------------------------------------------------------ */
/* Philox4x32-10 (Salmon et al., SC'11; the Random123 constants).  Reading Q7.          */
/* ------------------------------------------------------------------------------------ */
ODGR_API void odgr_philox4x32_10(const uint32_t ctr_in[4], const uint32_t key_in[2], uint32_t out[4]) {
  uint32_t c0 = ctr_in[0], c1 = ctr_in[1], c2 = ctr_in[2], c3 = ctr_in[3];
  uint32_t k0 = key_in[0], k1 = key_in[1];
  for (int round = 0; round < 10; ++round) {
    uint64_t prod0 = (uint64_t)0xD2511F53u * (uint64_t)c0;
    uint64_t prod1 = (uint64_t)0xCD9E8D57u * (uint64_t)c2;
    uint32_t hi0 = (uint32_t)(prod0 >> 32), lo0 = (uint32_t)prod0;
    uint32_t hi1 = (uint32_t)(prod1 >> 32), lo1 = (uint32_t)prod1;
    uint32_t n0 = hi1 ^ c1 ^ k0;
    uint32_t n1 = lo1;
    uint32_t n2 = hi0 ^ c3 ^ k1;
    uint32_t n3 = lo0;
    c0 = n0; c1 = n1; c2 = n2; c3 = n3;
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
  out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* u in (0,1) for candidate idx at iteration k on `stream` (0 = paths, 1 = trees).
 * u = ((r >> 9) + 1/2) * 2^-23: 23 random bits, exactly representable in fp32 (Q7). */
ODGR_API double odgr_uniform(uint64_t seed, uint64_t idx, uint64_t k, uint32_t stream) {
  uint32_t ctr[4] = {(uint32_t)(idx >> 2), (uint32_t)(idx >> 34), (uint32_t)k, stream};
  uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
  uint32_t r[4];
  odgr_philox4x32_10(ctr, key, r);
  uint32_t word = r[idx & 3];
  return ((double)(word >> 9) + 0.5) * (1.0 / 8388608.0);
}

/* g = -ln(-ln u), a Gumbel(0,1) sample (Jang et al. [16]). */
ODGR_API double odgr_gumbel(uint64_t seed, uint64_t idx, uint64_t k, uint32_t stream) {
  double u = odgr_uniform(seed, idx, k, stream);
  return -log(-log(u));
}

/* ------------------------------------------------------------------------------------ */
typedef struct {
  double a_wl, a_via, a_of;   /* a1, a2, a3 of Eq. (3): 0.5, 4, 500 */
  double beta;                /* beta_v of Eqs. (2)/(10) (reading Q3: global, default 0.25) */
  double n_layers;            /* L of Eq. (5)/(12) (reading Q4: 5) */
  int32_t f_kind;             /* 0 = sigmoid, 1 = ReLU, 2 = LeakyReLU, 3 = exp,
                                 4 = CELU (the alternatives of §5.3 / Fig. 6) */
  double f_slope;             /* sigmoid / exp: steepness s; LeakyReLU: negative slope; CELU: alpha (Q2) */
} odgr_weights;

typedef struct {
  int32_t X, Y;
  int64_t n_nets, n_trees, n_subnets, n_paths, n_segs, n_tps;
  int64_t *net_tree_off, *tree_sub_off, *sub_path_off, *path_seg_off, *path_tp_off;
  int32_t *seg, *tp_xy;
  real *cap_h, *cap_v;        /* [Y][X] */
  uint64_t seed;
  /* trainable logits and Adam state */
  real *w_tree, *w_path, *m_tree, *v_tree, *m_path, *v_path;
  int64_t *nid;               /* noise index of each path, -1 = none (reading Q7) */
  int64_t k;                  /* global iteration counter (noise key; Adam step = k+1) */
  int64_t net_lo, net_hi;     /* shard (all nets by default) */
  /* last forward */
  real *p, *q, *d_h, *d_v;
  real e_wl, e_tp, overflow, loss;
  double t_last;
} odgr_state;

static void* xcopy(const void* src, size_t bytes) {
  void* p = malloc(bytes ? bytes : 1);
  if (bytes) memcpy(p, src, bytes);
  return p;
}
static real* rzeros(size_t n) { return (real*)calloc(n + 1, sizeof(real)); }
static void to_double(double* dst, const real* src, size_t n) { for (size_t i = 0; i < n; ++i) dst[i] = (double)src[i]; }
static void to_real(real* dst, const double* src, size_t n) { for (size_t i = 0; i < n; ++i) dst[i] = (real)src[i]; }

ODGR_API int32_t odgr_real_bytes(void) { return (int32_t)sizeof(real); }

ODGR_API odgr_state* odgr_new(int32_t X, int32_t Y, int64_t n_nets, int64_t n_trees, int64_t n_subnets,
                              int64_t n_paths, int64_t n_segs, int64_t n_tps,
                              const int64_t* net_tree_off, const int64_t* tree_sub_off,
                              const int64_t* sub_path_off, const int64_t* path_seg_off,
                              const int64_t* path_tp_off, const int32_t* seg, const int32_t* tp_xy,
                              const float* cap_h, const float* cap_v, const float* w_tree0,
                              const float* w_path0, uint64_t seed) {
  odgr_state* s = (odgr_state*)calloc(1, sizeof(odgr_state));
  s->X = X; s->Y = Y;
  s->n_nets = n_nets; s->n_trees = n_trees; s->n_subnets = n_subnets; s->n_paths = n_paths;
  s->n_segs = n_segs; s->n_tps = n_tps;
  s->net_tree_off = (int64_t*)xcopy(net_tree_off, sizeof(int64_t) * (n_nets + 1));
  s->tree_sub_off = (int64_t*)xcopy(tree_sub_off, sizeof(int64_t) * (n_trees + 1));
  s->sub_path_off = (int64_t*)xcopy(sub_path_off, sizeof(int64_t) * (n_subnets + 1));
  s->path_seg_off = (int64_t*)xcopy(path_seg_off, sizeof(int64_t) * (n_paths + 1));
  s->path_tp_off = (int64_t*)xcopy(path_tp_off, sizeof(int64_t) * (n_paths + 1));
  s->seg = (int32_t*)xcopy(seg, sizeof(int32_t) * 4 * n_segs);
  s->tp_xy = (int32_t*)xcopy(tp_xy, sizeof(int32_t) * 2 * n_tps);
  size_t G = (size_t)X * Y;
  s->cap_h = rzeros(G);
  s->cap_v = rzeros(G);
  for (size_t e = 0; e < G; ++e) { s->cap_h[e] = cap_h[e]; s->cap_v[e] = cap_v[e]; }
  s->seed = seed;
  s->w_tree = rzeros(n_trees);
  s->w_path = rzeros(n_paths);
  for (int64_t j = 0; j < n_trees; ++j) s->w_tree[j] = w_tree0[j];
  for (int64_t i = 0; i < n_paths; ++i) s->w_path[i] = w_path0[i];
  /* Reading Q7: a sub-net whose only candidate is a straight path (one segment) draws no noise
   * (its softmax is 1 whatever the noise); every other candidate takes the next noise index. */
  s->nid = (int64_t*)malloc(sizeof(int64_t) * (n_paths + 1));
  int64_t next = 0;
  for (int64_t sn = 0; sn < n_subnets; ++sn) {
    int64_t i0 = sub_path_off[sn], i1 = sub_path_off[sn + 1];
    int lone_straight = (i1 - i0 == 1) && (path_seg_off[i0 + 1] - path_seg_off[i0] == 1);
    for (int64_t i = i0; i < i1; ++i) s->nid[i] = lone_straight ? -1 : next++;
  }
  s->m_tree = rzeros(n_trees); s->v_tree = rzeros(n_trees);
  s->m_path = rzeros(n_paths); s->v_path = rzeros(n_paths);
  s->p = rzeros(n_paths); s->q = rzeros(n_trees);
  s->d_h = rzeros(G); s->d_v = rzeros(G);
  s->k = 0;
  s->net_lo = 0; s->net_hi = n_nets;
  s->t_last = 1.0;
  return s;
}

ODGR_API void odgr_free(odgr_state* s) {
  if (!s) return;
  free(s->net_tree_off); free(s->tree_sub_off); free(s->sub_path_off); free(s->path_seg_off);
  free(s->path_tp_off); free(s->seg); free(s->tp_xy); free(s->cap_h); free(s->cap_v);
  free(s->nid);
  free(s->w_tree); free(s->w_path); free(s->m_tree); free(s->v_tree); free(s->m_path); free(s->v_path);
  free(s->p); free(s->q); free(s->d_h); free(s->d_v);
  free(s);
}

ODGR_API int64_t odgr_iteration(const odgr_state* s) { return s->k; }
ODGR_API void odgr_set_iteration(odgr_state* s, int64_t k) { s->k = k; }
/* restrict forward/backward/Adam to nets [lo,hi) — used only to test net sharding */
ODGR_API void odgr_set_shard(odgr_state* s, int64_t lo, int64_t hi) { s->net_lo = lo; s->net_hi = hi; }

/* WL_i: total length of i's segments in G-cell edges (reading Q5). TP_i: its turning points. */
static real path_wl(const odgr_state* s, int64_t i) {
  int64_t wl = 0;
  for (int64_t g = s->path_seg_off[i]; g < s->path_seg_off[i + 1]; ++g) wl += s->seg[4 * g + 3] - s->seg[4 * g + 2];
  return (real)wl;
}
static real path_tp(const odgr_state* s, int64_t i) { return (real)(s->path_tp_off[i + 1] - s->path_tp_off[i]); }

/* edge accessors: H edge (x,y)-(x+1,y) and V edge (x,y)-(x,y+1), both stored at [y][x] */
static real* edge_ref(real* gh, real* gv, int X, int dir, int line, int e) {
  return dir == 0 ? &gh[(size_t)line * X + e] : &gv[(size_t)e * X + line];
}

/* ---- forward, part 1 (this shard): probabilities and this shard's demand ---- */
/* p, q per §4.4; the demand of Eq. (10) added edge by edge; E[WL], E[TP] per Eqs. (11)/(12). */
static void forward_partial(odgr_state* s, real t, const odgr_weights* W, int noise, real* d_h, real* d_v,
                            real* e_wl, real* e_tp) {
  const int X = s->X, Y = s->Y;
  memset(d_h, 0, sizeof(real) * X * Y);
  memset(d_v, 0, sizeof(real) * X * Y);
  const real beta = (real)W->beta;
  real ewl = 0, etp = 0;
  for (int64_t n = s->net_lo; n < s->net_hi; ++n) {
    /* q_j = exp((w_j + g_j)/t) / sum_{k: net(k)=net(j)} exp((w_k + g_k)/t) */
    int64_t j0 = s->net_tree_off[n], j1 = s->net_tree_off[n + 1];
    real zmax = -INFINITY;
    for (int64_t j = j0; j < j1; ++j) {
      real g = noise ? (real)odgr_gumbel(s->seed, (uint64_t)j, (uint64_t)s->k, 1) : R(0);
      real z = (s->w_tree[j] + g) / t;
      s->q[j] = z;
      if (z > zmax) zmax = z;
    }
    real zs = 0;
    for (int64_t j = j0; j < j1; ++j) { s->q[j] = exp(s->q[j] - zmax); zs += s->q[j]; }
    for (int64_t j = j0; j < j1; ++j) s->q[j] /= zs;
    for (int64_t j = j0; j < j1; ++j) {
      for (int64_t sn = s->tree_sub_off[j]; sn < s->tree_sub_off[j + 1]; ++sn) {
        /* p_i = exp((w_i + g_i)/t) / sum_{k: subnet(k)=subnet(i)} exp((w_k + g_k)/t) */
        int64_t i0 = s->sub_path_off[sn], i1 = s->sub_path_off[sn + 1];
        real pm = -INFINITY;
        for (int64_t i = i0; i < i1; ++i) {
          real g = (noise && s->nid[i] >= 0) ? (real)odgr_gumbel(s->seed, (uint64_t)s->nid[i], (uint64_t)s->k, 0) : R(0);
          real z = (s->w_path[i] + g) / t;
          s->p[i] = z;
          if (z > pm) pm = z;
        }
        real ps = 0;
        for (int64_t i = i0; i < i1; ++i) { s->p[i] = exp(s->p[i] - pm); ps += s->p[i]; }
        for (int64_t i = i0; i < i1; ++i) s->p[i] /= ps;
        for (int64_t i = i0; i < i1; ++i) {
          real pi = s->q[j] * s->p[i];           /* q_tree(i) p_i */
          /* wire demand: every edge e of every segment of i */
          for (int64_t g = s->path_seg_off[i]; g < s->path_seg_off[i + 1]; ++g) {
            const int32_t* sg = &s->seg[4 * g];
            for (int e = sg[2]; e < sg[3]; ++e) *edge_ref(d_h, d_v, X, sg[0], sg[1], e) += pi;
          }
          /* via demand: beta * pi on every edge incident to each turning point v of i */
          for (int64_t u = s->path_tp_off[i]; u < s->path_tp_off[i + 1]; ++u) {
            int x = s->tp_xy[2 * u], y = s->tp_xy[2 * u + 1];
            real b = beta * pi;
            if (x >= 1) d_h[(size_t)y * X + (x - 1)] += b;
            if (x <= X - 2) d_h[(size_t)y * X + x] += b;
            if (y >= 1) d_v[(size_t)(y - 1) * X + x] += b;
            if (y <= Y - 2) d_v[(size_t)y * X + x] += b;
          }
          ewl += pi * path_wl(s, i);
          etp += pi * path_tp(s, i);
        }
      }
    }
  }
  *e_wl = ewl;
  *e_tp = etp;
}

ODGR_API void odgr_forward_partial(odgr_state* s, double t, const odgr_weights* W, int noise,
                                   double* d_h, double* d_v, double* e_wl, double* e_tp) {
  real ewl, etp;
  forward_partial(s, (real)t, W, noise, s->d_h, s->d_v, &ewl, &etp);
  to_double(d_h, s->d_h, (size_t)s->X * s->Y);
  to_double(d_v, s->d_v, (size_t)s->X * s->Y);
  *e_wl = (double)ewl;
  *e_tp = (double)etp;
}

static real sigm(real x) { return R(1) / (R(1) + exp(-x)); }

/* f applied to the resource r = cap - d, written in the overflow x = d - cap = -r (reading Q2):
 * sigmoid sigma(s x) = 1/(1+exp(s r)), ReLU max(0, x), LeakyReLU, exp(s x), CELU
 * (Fig. 6; torch conventions, negative slope / alpha in f_slope).  f_grad = df/dx = df/dd. */
static real f_of(int kind, real s, real x) {
  switch (kind) {
    case 0: return sigm(s * x);
    case 1: return x > 0 ? x : R(0);
    case 2: return x > 0 ? x : s * x;
    case 3: return exp(s * x);
    default: return x > 0 ? x : s * (exp(x / s) - R(1));
  }
}
static real f_grad(int kind, real s, real x) {
  switch (kind) {
    case 0: return s * sigm(s * x) * sigm(-s * x);
    case 1: return x > 0 ? R(1) : R(0);
    case 2: return x > 0 ? R(1) : s;
    case 3: return s * exp(s * x);
    default: return x > 0 ? R(1) : exp(x / s);
  }
}

/* ---- forward, part 2: the cost of Eq. (3) from the (global) demand in s->d_h, s->d_v ---- */
static real forward_finish(odgr_state* s, real e_wl, real e_tp, const odgr_weights* W, double out[4]) {
  const int X = s->X, Y = s->Y;
  const real slope = (real)W->f_slope;
  real of = 0;
  for (int y = 0; y < Y; ++y)
    for (int x = 0; x < X; ++x) {
      size_t e = (size_t)y * X + x;
      for (int dir = 0; dir < 2; ++dir) {
        if (dir == 0 && x > X - 2) continue;
        if (dir == 1 && y > Y - 2) continue;
        real r = (dir == 0 ? s->cap_h[e] - s->d_h[e] : s->cap_v[e] - s->d_v[e]);  /* resource */
        of += f_of(W->f_kind, slope, -r);
      }
    }
  s->e_wl = e_wl; s->e_tp = e_tp; s->overflow = of;
  real wl_cost = e_wl, via_cost = sqrt((real)W->n_layers) * e_tp;
  s->loss = (real)W->a_wl * wl_cost + (real)W->a_via * via_cost + (real)W->a_of * of;
  if (out) { out[0] = s->loss; out[1] = wl_cost; out[2] = via_cost; out[3] = of; }
  return s->loss;
}

ODGR_API double odgr_forward_finish(odgr_state* s, const double* d_h, const double* d_v, double e_wl,
                                    double e_tp, const odgr_weights* W, double out[4]) {
  to_real(s->d_h, d_h, (size_t)s->X * s->Y);
  to_real(s->d_v, d_v, (size_t)s->X * s->Y);
  return (double)forward_finish(s, (real)e_wl, (real)e_tp, W, out);
}

ODGR_API double odgr_forward(odgr_state* s, double t, const odgr_weights* W, int noise, double out[4]) {
  real ewl, etp;
  forward_partial(s, (real)t, W, noise, s->d_h, s->d_v, &ewl, &etp);
  s->t_last = t;
  return (double)forward_finish(s, ewl, etp, W, out);
}

/* ---- reverse: d cost / d w for the shard's logits (the chain rule of P:841-845) ---- */
static void backward(odgr_state* s, real t, const odgr_weights* W, real* dw_path, real* du_tree, real* c_path) {
  const int X = s->X, Y = s->Y;
  size_t G = (size_t)X * Y;
  const real a3 = (real)W->a_of, slope = (real)W->f_slope, beta = (real)W->beta;
  /* G_e = d cost / d d_e = -a3 f'(cap_e - d_e) */
  real* gh = rzeros(G);
  real* gv = rzeros(G);
  for (int y = 0; y < Y; ++y)
    for (int x = 0; x < X; ++x) {
      size_t e = (size_t)y * X + x;
      if (x <= X - 2) gh[e] = a3 * f_grad(W->f_kind, slope, s->d_h[e] - s->cap_h[e]);
      if (y <= Y - 2) gv[e] = a3 * f_grad(W->f_kind, slope, s->d_v[e] - s->cap_v[e]);
    }
  const real sqL = sqrt((real)W->n_layers);
  for (int64_t n = s->net_lo; n < s->net_hi; ++n) {
    int64_t j0 = s->net_tree_off[n], j1 = s->net_tree_off[n + 1];
    for (int64_t j = j0; j < j1; ++j) {
      real dq = 0;                      /* dq_j = sum_{i: tree(i)=j} p_i c_i */
      for (int64_t sn = s->tree_sub_off[j]; sn < s->tree_sub_off[j + 1]; ++sn) {
        int64_t i0 = s->sub_path_off[sn], i1 = s->sub_path_off[sn + 1];
        real spd = 0;                   /* sum_{k in subnet} p_k dp_k */
        for (int64_t i = i0; i < i1; ++i) {
          /* c_i = d cost / d pi_i */
          real c = (real)W->a_wl * path_wl(s, i) + (real)W->a_via * sqL * path_tp(s, i);
          for (int64_t g = s->path_seg_off[i]; g < s->path_seg_off[i + 1]; ++g) {
            const int32_t* sg = &s->seg[4 * g];
            for (int e = sg[2]; e < sg[3]; ++e) c += *edge_ref(gh, gv, X, sg[0], sg[1], e);
          }
          for (int64_t u = s->path_tp_off[i]; u < s->path_tp_off[i + 1]; ++u) {
            int x = s->tp_xy[2 * u], y = s->tp_xy[2 * u + 1];
            real v = 0;
            if (x >= 1) v += gh[(size_t)y * X + (x - 1)];
            if (x <= X - 2) v += gh[(size_t)y * X + x];
            if (y >= 1) v += gv[(size_t)(y - 1) * X + x];
            if (y <= Y - 2) v += gv[(size_t)y * X + x];
            c += beta * v;
          }
          if (c_path) c_path[i] = c;      /* (tests: the resolution of the gradient's fp32 evaluation) */
          dw_path[i] = s->q[j] * c;       /* dp_i = q_tree(i) c_i (stored temporarily) */
          dq += s->p[i] * c;
          spd += s->p[i] * dw_path[i];
        }
        /* softmax backward: dw_i = (p_i / t) (dp_i - sum_k p_k dp_k) */
        for (int64_t i = i0; i < i1; ++i) dw_path[i] = s->p[i] / t * (dw_path[i] - spd);
      }
      du_tree[j] = dq;
    }
    real sqd = 0;
    for (int64_t j = j0; j < j1; ++j) sqd += s->q[j] * du_tree[j];
    for (int64_t j = j0; j < j1; ++j) du_tree[j] = s->q[j] / t * (du_tree[j] - sqd);
  }
  free(gh);
  free(gv);
}

/* c_path (nullable): the per-candidate cost c_i = d cost / d pi_i of the same pass */
ODGR_API void odgr_backward_c(odgr_state* s, double t, const odgr_weights* W, double* dw_path, double* du_tree,
                              double* c_path) {
  real* dw = rzeros(s->n_paths);
  real* du = rzeros(s->n_trees);
  real* c = c_path ? rzeros(s->n_paths) : NULL;
  backward(s, (real)t, W, dw, du, c);
  for (int64_t n = s->net_lo; n < s->net_hi; ++n)
    for (int64_t j = s->net_tree_off[n]; j < s->net_tree_off[n + 1]; ++j) {
      du_tree[j] = du[j];
      for (int64_t i = s->sub_path_off[s->tree_sub_off[j]]; i < s->sub_path_off[s->tree_sub_off[j + 1]]; ++i) {
        dw_path[i] = dw[i];
        if (c) c_path[i] = c[i];
      }
    }
  free(dw);
  free(du);
  free(c);
}

ODGR_API void odgr_backward(odgr_state* s, double t, const odgr_weights* W, double* dw_path, double* du_tree) {
  odgr_backward_c(s, t, W, dw_path, du_tree, NULL);
}

/* ---- Adam (torch.optim.Adam semantics; betas 0.9/0.999, eps 1e-8; reading Q9) ---- */
static void adam_one(real* w, real* m, real* v, real g, real lr, int64_t step) {
  const real b1 = R(0.9), b2 = R(0.999), eps = R(1e-8);
  *m = b1 * *m + (R(1) - b1) * g;
  *v = b2 * *v + (R(1) - b2) * g * g;
  real bc1 = R(1) - pow(b1, (real)step), bc2 = R(1) - pow(b2, (real)step);
  real denom = sqrt(*v) / sqrt(bc2) + eps;
  *w -= (lr / bc1) * (*m / denom);
}

static void adam(odgr_state* s, real lr, const real* dw_path, const real* du_tree) {
  int64_t step = s->k + 1;
  for (int64_t n = s->net_lo; n < s->net_hi; ++n)
    for (int64_t j = s->net_tree_off[n]; j < s->net_tree_off[n + 1]; ++j) {
      adam_one(&s->w_tree[j], &s->m_tree[j], &s->v_tree[j], du_tree[j], lr, step);
      for (int64_t sn = s->tree_sub_off[j]; sn < s->tree_sub_off[j + 1]; ++sn)
        for (int64_t i = s->sub_path_off[sn]; i < s->sub_path_off[sn + 1]; ++i)
          adam_one(&s->w_path[i], &s->m_path[i], &s->v_path[i], dw_path[i], lr, step);
    }
}

ODGR_API void odgr_adam(odgr_state* s, double lr, const double* dw_path, const double* du_tree) {
  real* dw = rzeros(s->n_paths);
  real* du = rzeros(s->n_trees);
  to_real(dw, dw_path, (size_t)s->n_paths);
  to_real(du, du_tree, (size_t)s->n_trees);
  adam(s, (real)lr, dw, du);
  free(dw);
  free(du);
}

ODGR_API void odgr_next_iteration(odgr_state* s) { s->k += 1; }

/* iters x {forward, reverse, Adam}; iters = 0 is forward only (include/dgr.h contract) */
ODGR_API void odgr_step(odgr_state* s, int iters, double t, double lr, const odgr_weights* W, double out[4]) {
  if (iters == 0) { odgr_forward(s, t, W, 1, out); return; }
  real* dw = rzeros(s->n_paths);
  real* du = rzeros(s->n_trees);
  for (int it = 0; it < iters; ++it) {
    odgr_forward(s, t, W, 1, out);
    backward(s, (real)t, W, dw, du, NULL);
    adam(s, (real)lr, dw, du);
    s->k += 1;
  }
  free(dw);
  free(du);
}

ODGR_API void odgr_get_logits(const odgr_state* s, double* w_tree, double* w_path) {
  if (w_tree) to_double(w_tree, s->w_tree, (size_t)s->n_trees);
  if (w_path) to_double(w_path, s->w_path, (size_t)s->n_paths);
}
ODGR_API void odgr_set_logits(odgr_state* s, const double* w_tree, const double* w_path) {
  if (w_tree) to_real(s->w_tree, w_tree, (size_t)s->n_trees);
  if (w_path) to_real(s->w_path, w_path, (size_t)s->n_paths);
}
ODGR_API void odgr_get_adam(const odgr_state* s, double* m_tree, double* v_tree, double* m_path, double* v_path) {
  if (m_tree) to_double(m_tree, s->m_tree, (size_t)s->n_trees);
  if (v_tree) to_double(v_tree, s->v_tree, (size_t)s->n_trees);
  if (m_path) to_double(m_path, s->m_path, (size_t)s->n_paths);
  if (v_path) to_double(v_path, s->v_path, (size_t)s->n_paths);
}
ODGR_API void odgr_get_probs(const odgr_state* s, double* q, double* p) {
  if (q) to_double(q, s->q, (size_t)s->n_trees);
  if (p) to_double(p, s->p, (size_t)s->n_paths);
}
ODGR_API void odgr_get_demand(const odgr_state* s, double* d_h, double* d_v) {
  to_double(d_h, s->d_h, (size_t)s->X * s->Y);
  to_double(d_v, s->d_v, (size_t)s->X * s->Y);
}

/* ---- discrete induction (§4.5; readings Q12, Q13, Q23) ----
 * p_hat, q_hat = noise-free softmax(w / t_final).  tree* = argmax q_hat (ties: lowest index).
 * For each sub-net of tree*: rank its paths by p_hat descending (ties: lowest index) and keep
 * the smallest prefix whose cumulative p_hat reaches top_p (at least one path); the route is the
 * first path of that prefix.  Sub-nets of unchosen trees get route = -1 and an empty nucleus.
 * D = integer wire demand of the routes (Eq. (2)'s first term with one-hot x, y);
 * metrics = {sum_e max(0, D_e + beta V_e - cap_e), #edges with that > 0, its maximum,
 *            sum WL of routes, sum TP of routes}, V_e = route turning points incident to e.
 * margins (optional): per net the q_hat gap top1 - top2; per sub-net the p_hat gap top1 - top2
 * and min_r |cumsum_r - top_p| over the ranks up to the nucleus end (1 when undefined). */
ODGR_API void odgr_induce(const odgr_state* s, double t_final, double top_p, double beta,
                          int32_t* tree_choice, int32_t* route, int64_t* nucleus_off, int32_t* nucleus,
                          int32_t* D_h, int32_t* D_v, double metrics[5], double* margin_tree,
                          double* margin_route, double* margin_nucleus) {
  const int X = s->X, Y = s->Y;
  memset(D_h, 0, sizeof(int32_t) * X * Y);
  memset(D_v, 0, sizeof(int32_t) * X * Y);
  int32_t* V = (int32_t*)calloc((size_t)X * Y, sizeof(int32_t));  /* route turning points per G-cell */
  double sum_wl = 0, sum_tp = 0;
  int64_t nn = 0;
  nucleus_off[0] = 0;
  for (int64_t n = 0; n < s->n_nets; ++n) {
    int64_t j0 = s->net_tree_off[n], j1 = s->net_tree_off[n + 1];
    /* q_hat over the net's trees */
    double zmax = -INFINITY;
    for (int64_t j = j0; j < j1; ++j) if (s->w_tree[j] / t_final > zmax) zmax = s->w_tree[j] / t_final;
    double zs = 0;
    for (int64_t j = j0; j < j1; ++j) zs += exp(s->w_tree[j] / t_final - zmax);
    int64_t best = j0;
    double qb = -1, q2 = -1;
    for (int64_t j = j0; j < j1; ++j) {
      double qj = exp(s->w_tree[j] / t_final - zmax) / zs;
      if (qj > qb) { q2 = qb; qb = qj; best = j; }
      else if (qj > q2) q2 = qj;
    }
    tree_choice[n] = (int32_t)best;
    if (margin_tree) margin_tree[n] = (j1 - j0 > 1) ? qb - q2 : 1.0;
    for (int64_t j = j0; j < j1; ++j) {
      for (int64_t sn = s->tree_sub_off[j]; sn < s->tree_sub_off[j + 1]; ++sn) {
        int64_t i0 = s->sub_path_off[sn], i1 = s->sub_path_off[sn + 1];
        int64_t m = i1 - i0;
        if (j != best) {
          route[sn] = -1;
          nucleus_off[sn + 1] = nn;
          if (margin_route) margin_route[sn] = 1.0;
          if (margin_nucleus) margin_nucleus[sn] = 1.0;
          continue;
        }
        double* ph = (double*)malloc(sizeof(double) * m);
        int64_t* ord = (int64_t*)malloc(sizeof(int64_t) * m);
        double pm = -INFINITY, ps = 0;
        for (int64_t a = 0; a < m; ++a) if (s->w_path[i0 + a] / t_final > pm) pm = s->w_path[i0 + a] / t_final;
        for (int64_t a = 0; a < m; ++a) { ph[a] = exp(s->w_path[i0 + a] / t_final - pm); ps += ph[a]; }
        for (int64_t a = 0; a < m; ++a) { ph[a] /= ps; ord[a] = a; }
        /* insertion sort by (p_hat desc, index asc) */
        for (int64_t a = 1; a < m; ++a) {
          int64_t key = ord[a], b = a - 1;
          while (b >= 0 && (ph[ord[b]] < ph[key] || (ph[ord[b]] == ph[key] && ord[b] > key))) { ord[b + 1] = ord[b]; --b; }
          ord[b + 1] = key;
        }
        double cum = 0, mn = 1.0;
        int64_t r = 0;
        for (; r < m; ++r) {
          if (r > 0 && cum >= top_p) break;     /* stop once the prefix reached top_p */
          cum += ph[ord[r]];
          double gap = fabs(cum - top_p);
          if (gap < mn) mn = gap;
          nucleus[nn++] = (int32_t)(i0 + ord[r]);
        }
        nucleus_off[sn + 1] = nn;
        route[sn] = (int32_t)(i0 + ord[0]);
        if (margin_route) margin_route[sn] = m > 1 ? ph[ord[0]] - ph[ord[1]] : 1.0;
        if (margin_nucleus) margin_nucleus[sn] = mn;
        int64_t i = i0 + ord[0];
        for (int64_t g = s->path_seg_off[i]; g < s->path_seg_off[i + 1]; ++g) {
          const int32_t* sg = &s->seg[4 * g];
          for (int e = sg[2]; e < sg[3]; ++e) {
            if (sg[0] == 0) D_h[(size_t)sg[1] * X + e] += 1;
            else D_v[(size_t)e * X + sg[1]] += 1;
          }
        }
        for (int64_t u = s->path_tp_off[i]; u < s->path_tp_off[i + 1]; ++u)
          V[(size_t)s->tp_xy[2 * u + 1] * X + s->tp_xy[2 * u]] += 1;
        sum_wl += path_wl(s, i);
        sum_tp += path_tp(s, i);
        free(ph);
        free(ord);
      }
    }
  }
  double tot = 0, mx = 0;
  int64_t cnt = 0;
  for (int y = 0; y < Y; ++y)
    for (int x = 0; x < X; ++x) {
      size_t e = (size_t)y * X + x;
      if (x <= X - 2) {
        double o = D_h[e] + beta * (V[e] + V[e + 1]) - s->cap_h[e];
        if (o > 0) { tot += o; cnt++; if (o > mx) mx = o; }
      }
      if (y <= Y - 2) {
        double o = D_v[e] + beta * (V[e] + V[e + X]) - s->cap_v[e];
        if (o > 0) { tot += o; cnt++; if (o > mx) mx = o; }
      }
    }
  metrics[0] = tot; metrics[1] = (double)cnt; metrics[2] = mx; metrics[3] = sum_wl; metrics[4] = sum_tp;
  free(V);
}
