/* dgr.h — C ABI of libdgr: the B200 (sm_100a) DGR differentiable DAG-forest solver.
 *
 * The operation: PAPER.md (DGR, DAC'24) §4.3-4.5.  One solver iteration (dgr_step) is
 *   (1) Gumbel-softmax over every net's routing-tree candidates and every 2-pin sub-net's
 *       path candidates                                      §4.4
 *   (2) expected demand on the H/V G-cell edges, Eq. (10)
 *   (3) cost = a1 WL + a2 via + a3 overflow, Eqs. (9),(11),(12)
 *   (4) its gradient w.r.t. the logits (the paper uses autograd)
 *   (5) Adam on the logits
 * and dgr_induce is the discrete selection of §4.5 (argmax tree, top-p paths).
 * The readings of the paper this library implements are listed in DESIGN.md §3
 * (grouping = sub-net, f of the overflow x = d - cap, beta_v global, sqrt(L) with L = n_layers,
 * Philox4x32-10 noise keyed on (seed, noise index, iteration, stream); see dgr_forest_desc).
 *
 * Conventions for every entry point
 *   - return int: 0 = DGR_OK, < 0 = error code below; dgr_last_error() (thread-local) says why.
 *     No C++ exception crosses this boundary.  An error leaves no partial state behind.
 *   - host pointers are caller-owned, read during the call only (inputs are copied at load).
 *   - the device workspace is caller-owned memory (e.g. a torch uint8 CUDA tensor) of at least
 *     dgr_workspace_size() bytes that must outlive the handle; its layout is library-owned.
 *   - all work is ordered on the cudaStream_t passed to dgr_forest_load; calls that return
 *     data to the host synchronise that stream.
 *   - a handle is not thread-safe.  With world > 1 there is one process per GPU, each with its
 *     own handle, and dgr_step / dgr_induce are collective over the ranks (NCCL).
 *
 * Geometry (identical to include/forestgen.h)
 *   G-cell grid X x Y.  H edge (x,y)-(x+1,y), x in [0,X-2]; V edge (x,y)-(x,y+1), y in [0,Y-2].
 *   Grids are row-major [Y][X]; the last column (H) / last row (V) is padding.
 *   Segment {dir (0 = H, 1 = V), line (y for H, x for V), lo, hi}: the edges [lo,hi) of the line.
 *   A path candidate is any rectilinear path given as its segments and turning points (§3.1,
 *   L-, Z-, C-shape patterns and monotonic routes); each sub-net has 1..1024.
 */
#ifndef DGR_H
#define DGR_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

enum {
  DGR_OK = 0,
  DGR_EINVAL = -1,   /* invalid argument or malformed forest (nothing was allocated or changed) */
  DGR_ECUDA = -2,    /* a CUDA runtime call failed */
  DGR_ENCCL = -3,    /* an NCCL call failed */
  DGR_ENOMEM = -4,   /* workspace too small / host allocation failed */
  DGR_ESTATE = -5    /* call not valid in the handle's state (e.g. dgr_get_demand before a forward) */
};

/* Message of the last failed call on this thread; every entry point clears it first ("" = success). */
const char* dgr_last_error(void);

/* The routing DAG forest F = {T, S, P} of §3.2 as flat CSR arrays, in GLOBAL order.
 * Offsets have length n+1, start at 0 and are non-decreasing; every group is non-empty.
 * Path candidates (§3.1) are rectilinear paths: every segment a non-empty edge range of
 * a grid line, every turning point a G-cell on one of the path's segments (else DGR_EINVAL).  A
 * sub-net whose candidates are its straight path, or HV, VH, Z-HVH..., Z-VHV..., C-shapes in that
 * order (the order forestgen emits), 32 at most, runs in the tile kernels; any other sub-net
 * (monotone staircases, other orders, up to 1024 candidates) makes its net run on the general
 * path (row f4': one warp per net over the explicit segment lists).  Same results
 * either way; the order of a sub-net's candidates is its tie-break order (induction).
 * Gumbel noise (Q7): a sub-net whose only candidate is a straight path draws none (its
 * softmax is identically 1); every other candidate, in global path order, takes the next noise
 * index n (0, 1, 2, ...) and draws g from Philox4x32-10(key = seed, counter = {n >> 2 (64 bit),
 * k, 0}) word n & 3; tree j draws from counter {j >> 2, k, 1} word j & 3. */
typedef struct {
  int32_t X, Y;                           /* grid; 2..32767 each */
  int64_t n_nets, n_trees, n_subnets, n_paths, n_segs, n_tps;
  const int64_t* net_tree_off;            /* net -> its routing-tree candidates (T) */
  const int64_t* tree_sub_off;            /* tree -> its 2-pin sub-nets (S) */
  const int64_t* sub_path_off;            /* sub-net -> its path candidates (P), 1..32 each */
  const int64_t* path_seg_off;            /* path -> its segments */
  const int64_t* path_tp_off;             /* path -> its turning points */
  const int32_t* seg;                     /* n_segs x {dir, line, lo, hi} */
  const int32_t* tp_xy;                   /* n_tps x {x, y} */
  const int32_t* sub_xy;                  /* n_subnets x {x0, y0, x1, y1} (either orientation) */
  const float* cap_h;                     /* [Y][X] capacity of H edges, Eq. (1) */
  const float* cap_v;                     /* [Y][X] capacity of V edges */
  const float* w_tree0;                   /* [n_trees] initial logits w */
  const float* w_path0;                   /* [n_paths] */
  uint64_t seed;                          /* Philox key of the Gumbel noise */
} dgr_forest_desc;

/* Caller-supplied exchange (optional, replaces NCCL): an in-place sum over the ranks of `count`
 * elements at device pointer `buf` (dtype 0 = int64, 1 = int32, 2 = fp64, 3 = fp32; the library
 * expresses its reduce-scatter / all-gather steps through it: all-gather zeroes the other ranks'
 * chunks first, so fp64 / fp32 sums are exact), ordered after the work already
 * enqueued on `cuda_stream` and visible to the work enqueued after the call returns.  Returns 0 on
 * success; any other value makes the calling dgr_* function fail with DGR_ENCCL.  Used to run
 * several ranks in one process (e.g. on one GPU, for testing the sharded path without NCCL). */
typedef int (*dgr_allreduce_fn)(void* user, void* buf, int64_t count, int32_t dtype, void* cuda_stream);

/* Multi-GPU: one process per GPU.  rank 0 calls dgr_nccl_unique_id and broadcasts the 128
 * bytes (e.g. over torch.distributed); every rank passes them here. NULL, or world == 1 with
 * neither an id nor a callback: single GPU, no exchange.  world == 1 WITH an NCCL id (or a
 * callback) runs the band exchange of world > 1 through a one-rank communicator (or the callback):
 * the same results, the NCCL path exercised on one GPU (tests).
 * With `allreduce` non-NULL the ranks exchange through it instead (nccl_unique_id unused). */
typedef struct {
  int32_t rank, world;
  const void* nccl_unique_id;             /* 128 bytes */
  dgr_allreduce_fn allreduce;             /* NULL: NCCL */
  void* allreduce_user;
} dgr_dist;

/* Cost weights and model constants. */
typedef struct {
  float a_wl, a_via, a_of;   /* a1, a2, a3 of Eq. (3); paper: 0.5, 4, 500 */
  float beta_via;            /* beta_v of Eqs. (2)/(10), one global value (Q3; default 0.25) */
  float n_layers;            /* L in sqrt(L) of Eqs. (5)/(12) (Q4; default 5) */
  int32_t f_kind;            /* overflow function f of Eq. (9) of x = d - cap (Q2): 0 = sigmoid(s x)
                                (P:912), 1 = ReLU, 2 = LeakyReLU, 3 = exp(s x), 4 = CELU
                                (the alternatives studied in Fig. 6) */
  float f_slope;             /* sigmoid / exp: s (default 1); LeakyReLU: negative slope (0.01); CELU: alpha (1) */
} dgr_weights;

/* Loss of a forward pass: total = a_wl*wl + a_via*via + a_of*overflow, with
 * wl = E[WL] (Eq. 11), via = sqrt(L) E[TP] (Eq. 12), overflow = sum_e f(d_e - cap_e) (Eq. 9), f of
 * the overflow x = d - cap (reading Q2: the paper's f(cap - d) with f decreasing). */
typedef struct { double total, wl, via, overflow; } dgr_loss;

struct dgr_handle;

/* Writes the 128-byte ncclUniqueId (call on rank 0 only). */
int dgr_nccl_unique_id(void* out128);

/* Contiguous net ranges [out[r], out[r+1]) for `world` ranks, balanced on the candidate work
 * (paths + segments) of each net; out has world+1 entries.  Host-only, no GPU needed. */
int dgr_partition(const dgr_forest_desc* desc, int32_t world, int64_t* out);

/* Bytes of device workspace this rank needs for desc (0 on error; see dgr_last_error). */
int64_t dgr_workspace_size(const dgr_forest_desc* desc, const dgr_dist* dist);

/* Host-only first half of dgr_forest_load: validates desc, keeps this rank's nets (dgr_partition)
 * and encodes them (tiles, bundles; SURVEY §8(b) "forest encoding").  The handle owns the plan but
 * no device memory yet: only dgr_handle_workspace_size, dgr_bind_workspace, dgr_get_info and
 * dgr_free are valid on it (others return DGR_ESTATE).  cuda_stream as in dgr_forest_load. */
int dgr_forest_plan(const dgr_forest_desc* desc, const dgr_dist* dist, void* cuda_stream, struct dgr_handle** out);

/* Bytes of device workspace a planned handle needs (0 on error). */
int64_t dgr_handle_workspace_size(struct dgr_handle* h);

/* Second half of dgr_forest_load: copies the planned shard into dev_workspace (>= the planned
 * size, 256-byte aligned; caller-owned, must outlive the handle), zeroes Adam state and k and, with
 * world > 1, creates the NCCL communicator (collective).  desc and dist must describe the same
 * forest and ranks as at dgr_forest_plan (w_path0, w_tree0, cap_h, cap_v and seed are read here).
 * On error the handle stays planned (the caller may retry or free it).  Synchronises. */
int dgr_bind_workspace(struct dgr_handle* h, const dgr_forest_desc* desc, const dgr_dist* dist,
                       void* dev_workspace, int64_t workspace_bytes);

/* dgr_forest_plan + dgr_bind_workspace in one call (plans the forest once; dgr_workspace_size
 * above plans it separately).
 * Validates desc, keeps this rank's nets (dgr_partition), encodes them for the device, copies
 * them into dev_workspace (>= dgr_workspace_size bytes, 256-byte aligned) on cuda_stream
 * (a cudaStream_t; NULL = legacy default stream), zeroes Adam state and the iteration counter k.
 * With world > 1 this also creates the NCCL communicator (collective), unless dist->allreduce
 * supplies the exchange.  Synchronises. */
int dgr_forest_load(const dgr_forest_desc* desc, const dgr_dist* dist, void* dev_workspace,
                    int64_t workspace_bytes, void* cuda_stream, struct dgr_handle** out);

/* Runs `iters` solver iterations at temperature t and Adam learning rate lr: each is
 * forward (steps 1-3), reverse (step 4) and Adam (step 5), with k incremented after each.
 * iters == 0 runs one forward only (no update, k unchanged).  The Gumbel noise of iteration k
 * is keyed on the global k, so 10 calls of 100 iterations equal 1 call of 1000 at equal t.
 * The last iteration also runs the forward of iteration k+1 (device-side state only), so a
 * following call at the same temperature starts from it instead of recomputing it. 
 * If `last` is non-NULL it receives the loss of the last forward (synchronises). */
int dgr_step(struct dgr_handle* h, int32_t iters, float temperature, float lr, const dgr_weights* w,
             dgr_loss* last);

/* dgr_step without host synchronisation (the same iterations of PAPER.md §4.3-4.4, P:803-847,
 * P:913-914), then a stream-ordered write of the
 * loss of the last forward (4 doubles: total, wl, via, overflow, as dgr_loss) into loss_out
 * (host memory, caller-owned): pinned (page-locked, device-accessible) memory is written by the
 * loss kernel itself, with no copy on the stream; pageable memory gets a cudaMemcpyAsync after it.
 * loss_out is valid after dgr_sync or any synchronising call on the handle.  NULL loss_out:
 * DGR_EINVAL. */
int dgr_step_async(struct dgr_handle* h, int32_t iters, float temperature, float lr, const dgr_weights* w,
                   double* loss_out);

/* Waits for all work the handle has enqueued on its stream. */
int dgr_sync(struct dgr_handle* h);

/* Demand d_e (Eq. 10) of the last forward, full grids [Y][X] (H padding column / V padding
 * row are 0).  With world > 1 this is the global (all-rank) demand.  Synchronises. */
int dgr_get_demand(struct dgr_handle* h, float* d_h, float* d_v);

/* Current logits in GLOBAL order.  With world > 1 only this rank's entries are written. */
int dgr_get_logits(struct dgr_handle* h, float* w_tree, float* w_path);

/* Discrete selection of §4.5 from the current logits at the temperature of the last dgr_step
 * (noise-free softmax): tree_choice[n] = global index of argmax_j q_hat (ties: lowest index);
 * for each sub-net of a chosen tree the paths ranked by p_hat descending (ties: lowest index),
 * the nucleus = the smallest prefix whose cumulative p_hat reaches top_p (at least one path),
 * route[s] = its first path (global index), -1 for sub-nets of unchosen trees.
 * nucleus_off [n_subnets+1] / nucleus (capacity n_paths) hold the nuclei as CSR in sub-net order.
 * D_h, D_v [Y][X]: integer wire demand of the routes; metrics = {sum_e max(0, D_e + beta V_e -
 * cap_e), number of edges where that is > 0, its maximum, sum WL, sum TP} of the routes, V_e =
 * route turning points at e's end cells.  With world > 1, entries outside this rank's nets are
 * -1 / empty and D_h, D_v, metrics are global.  Synchronises. */
int dgr_induce(struct dgr_handle* h, float top_p, int32_t* tree_choice, int32_t* route,
               int64_t* nucleus_off, int32_t* nucleus, int32_t* D_h, int32_t* D_v, double metrics[5]);

/* Introspection: iteration counter k, this rank's net range, encoded sizes.  info[12] =
 * {k, net_lo, net_hi, n_bundles, n_path_slots, workspace_bytes, world, rank, n_tiles,
 *  n_global_tiles, n_pipelined_tiles, n_general_paths} (candidates on the general path). */
int dgr_get_info(struct dgr_handle* h, int64_t info[12]);

/* Host-only view of the rank's encoding plan (no GPU needed): out[8] = {n_tiles, n_global_tiles,
 * n_bundles, n_path_slots, workspace_bytes, n_paths, paths in global tiles, largest window (cells)}.
 * A tile is a run of whole nets whose candidates fit one shared-memory window of the grid; a
 * global tile's nets are too spread out and run against HBM directly. */
int dgr_plan_info(const dgr_forest_desc* desc, const dgr_dist* dist, int64_t out[8]);

/* Per-stage device time of subsequent dgr_step calls, from CUDA events recorded on the handle's
 * stream after every stage.  enable != 0 starts (and clears) recording, 0 stops it.
 * dgr_profile_read synchronises and returns, per stage, the summed milliseconds and the number of
 * launches: 0 KF (forward-only tile kernel, once per dgr_step call), 1 demand allreduce (NCCL;
 * world > 1), 2 KG (scan / loss / gradient map; 1 kernel), 3 KBF (reverse of k fused with the
 * forward of k+1), 4 KB (reverse only; not launched since every call ends with KBF), 5 KL (the loss reduction,
 * once per call after its last KG), 6..7 unused. */
int dgr_profile(struct dgr_handle* h, int32_t enable);
int dgr_profile_read(struct dgr_handle* h, double ms[8], int64_t launches[8]);

/* Releases the handle (and the NCCL communicator); the workspace stays the caller's. */
int dgr_free(struct dgr_handle* h);

/* ---------------------------------------------------------------------------------------------
 * Row f1: routing-DAG-forest construction on the GPU, one thread per net (§4.2; the
 * paper leaves it to "net-level parallelism").  Readings: tree
 * candidates Q17 (Prim MST from pin 0; iterated 1-Steiner on the Hanan grid for <= 8 pins, else
 * Prim from the last pin; a duplicate second candidate is dropped), sub-nets = tree edges in Prim
 * order with canonical endpoints, paths Q14 (straight, or HV, VH, z_cap-limited Z-HVH / Z-VHV, then
 * c_cap C-HVH / C-VHV detours per side, Q14b),
 * initial logits Q8 (U[0,1), splitmix64 counter hash of (seed, 3 / 4, index)).  The result equals
 * forestgen's forest for the same pins, bit for bit.
 * ------------------------------------------------------------------------------------------- */
typedef struct {
  int32_t X, Y;                 /* grid, 2..32767 per side */
  int64_t n_nets;
  const int64_t* net_pin_off;   /* [n_nets+1] host */
  const int32_t* pin_xy;        /* [n_pins][2] host; 2..32 distinct in-grid pins per net */
  int32_t n_tree_cand;          /* 1 or 2 */
  int32_t z_cap;                /* -1: L only; 0: every Z; > 0: at most z_cap Z per direction */
  uint64_t seed;                /* of the initial logits */
  int32_t c_cap;                /* C-shape detours per side of a non-aligned sub-net (0 = none; Q14b, row f4) */
} dgr_pins_desc;

struct dgr_built_forest;

/* Builds the forest on cuda_stream into device memory owned by the returned object
 * (cudaMallocAsync; released by dgr_built_forest_free).  Pins are read during the call only.
 * Synchronises (the output sizes are data-dependent).  DGR_EINVAL for malformed pins. */
int dgr_build_forest(const dgr_pins_desc* pins, void* cuda_stream, struct dgr_built_forest** out);

/* sizes = {nets, trees, sub-nets, paths, segments, turning points} */
int dgr_built_forest_sizes(const struct dgr_built_forest* f, int64_t sizes[6]);

/* Copies the forest into caller-owned host arrays shaped like dgr_forest_desc's (any may be NULL
 * to skip it).  Synchronises. */
int dgr_built_forest_download(const struct dgr_built_forest* f, int64_t* net_tree_off, int64_t* tree_sub_off,
                              int64_t* sub_path_off, int64_t* path_seg_off, int64_t* path_tp_off,
                              int32_t* sub_xy, int32_t* seg, int32_t* tp_xy, float* w_tree0, float* w_path0);

int dgr_built_forest_free(struct dgr_built_forest* f);

#ifdef __cplusplus
}
#endif
#endif
