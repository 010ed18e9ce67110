// dgr_internal.h — device data layout shared by the libdgr host code and its sm_100a kernels.
//
// Layout in HBM:
//   * candidates live in 32-slot "bundles": one warp processes one bundle, one lane one path
//     candidate.  A "group" bundle holds whole sub-nets (groups of 1..32 candidates, packed in
//     order, never split), so the sub-net softmax is a segmented warp reduction.  Sub-nets whose
//     only candidate is a straight path ("singletons": p = 1 identically, no logit update) are
//     packed 32 to a "singleton" bundle and skip noise, softmax and Adam.  Unused tail lanes are
//     padding (shape PAD).
//   * bundles are grouped into "tiles": whole nets whose candidates all lie inside one small
//     G-cell window (<= kWinMax cells incl. a 1-cell halo).  One CTA owns one tile: it stages the
//     tile's window of the gradient prefix sums in shared memory for the reverse pass, keeps the
//     tile's tree state (dq, q) in shared memory, and accumulates the tile's demand events in a
//     shared-memory window that it flushes once to the global difference arrays.  Tiles whose
//     nets span a larger window run the same code against global memory ("global" tiles).
//     A tile's bundles are its group bundles, then its singleton bundles; its sub-nets are stored
//     in that "kernel order" too (a permutation of the tile's sub-net range).
//   * per slot:    pword (shape | flags | tree offset | mid), w, m, v (fp32), p of the last
//     forward (fp32)
//   * per bundle:  {tile noise offset of lane 0 (its noisy candidates before this bundle), first
//     kernel-order sub-net, the tile's first tree, #valid lanes | kSingleBundle}
//   * per sub-net: canonical endpoints (x0 <= x1; y0 < y1 if x0 == x1) as int16 x 4
//   * per tree:    w, m, v, q (fp32)
//   * grids: difference arrays of the demand along H rows ([Y][X]) and along V columns (stored
//     transposed, [X][Y], so both scans run over contiguous lines), int64 in 2^-40 fixed point,
//     with each turning point's beta pi folded in as a +-beta pi window over its incident edges
//     (Eq. (10), reading Q3), followed by two int64 counters (E[TP] and a border term, 2^-24) of
//     the same forward: this is the whole per-iteration exchange buffer; prefix sums S of the
//     overflow gradient per line (fp64, the same two layouts).
#pragma once
#include <cstdint>

namespace dgr {

constexpr int kFracBits = 24;                      // fixed point of pi: round(pi * 2^24)
constexpr float kFixScale = 16777216.0f;           // 2^24
constexpr double kFixInv = 1.0 / 16777216.0;
constexpr int kGridShift = 16;                     // difference arrays: 2^-(24+16) = 2^-40 fixed point
constexpr double kGridInv = 1.0 / 1099511627776.0; // 2^-40
constexpr double kGridBeta = 65536.0;              // beta pi (pi in 2^-24) -> 2^-40: exact for beta in 2^-16 Z
constexpr double kDqScale = 4294967296.0;          // dq_j accumulated in 2^-32 fixed point
constexpr double kDqInv = 1.0 / 4294967296.0;

constexpr int kTileThreads = 256;                  // 8 warps per tile CTA
#ifndef DGR_WINMAX
#define DGR_WINMAX 1536
#endif
constexpr int kWinMax = DGR_WINMAX;                // window cells per tile
constexpr int kMaxBundles = 64;                    // bundles per tile (a whole net always fits)
#ifndef DGR_TARGET_BUNDLES
#define DGR_TARGET_BUNDLES 32
#endif
constexpr int kTargetBundles = DGR_TARGET_BUNDLES;  // group bundles per pipelined tile
constexpr int kTileBundles = kTargetBundles + 8;   // all bundles (group + singleton) per pipelined tile
constexpr int kTreeMax = 512;                      // trees per tile
#ifndef DGR_PIPE_TREES
#define DGR_PIPE_TREES 224
#endif
constexpr int kPipeTrees = DGR_PIPE_TREES;         // trees per pipelined tile
#ifndef DGR_PIPE_SUBS
#define DGR_PIPE_SUBS 512
#endif
constexpr int kPipeSubs = DGR_PIPE_SUBS;           // sub-nets per pipelined tile
#ifndef DGR_KG_WARPS
#define DGR_KG_WARPS 8
#endif
constexpr int kKgWarps = DGR_KG_WARPS;             // warps per KG CTA (one line per CTA)
constexpr int kEventMax = 127;                     // events per window cell-field (int32 safety)
constexpr int kGenMaxGroup = 1024;                 // candidates per sub-net (general path, row f4')
constexpr int kGenWarps = 8;                       // general nets per CTA (one warp each)

enum Shape : uint32_t {
  kStraightH = 0, kStraightV = 1, kHV = 2, kVH = 3, kZHVH = 4, kZVHV = 5, kPad = 7
};
constexpr uint32_t kSubHead = 8u;    // lane starts a sub-net group
constexpr uint32_t kTreeHead = 16u;  // group head whose tree differs from the previous group's in the bundle
constexpr int kTreeShift = 5;        // bits 5..13: tree of the lane relative to the bundle's tree base
constexpr uint32_t kTreeMask = 511u;
constexpr uint32_t kMultiTree = 1u << 15; // the candidate's net has >= 2 trees: its tree's dq is used
                                           // (a lone tree has du = 0, so its dq is never needed)
constexpr uint32_t kOutside = 1u << 14;   // Z-HVH / Z-VHV shape whose x_m / y_m lies outside the
                                           // sub-net's span: a C-shape detour (row f4, reading Q14b)
// bits 16..31: x_m (Z-HVH) or y_m (Z-VHV)
constexpr int kSingleBundle = 0x100; // binfo.w flag: a singleton bundle (binfo.w & 0xff = #valid)

struct TileDesc {
  int32_t b0, nb;          // bundles [b0, b0 + nb)
  int32_t net0, nnet;      // local nets
  int32_t tree0, ntree;    // local trees
  int32_t wx0, wy0, ww, wh;  // window (cells; even origin and extents), unused for global tiles
  int32_t global, nbg;     // nbg: group bundles (the first nbg of the tile; the rest are singleton bundles)
  int32_t sub0, nsub;      // local sub-nets (kernel order within the tile)
  int32_t mn0, nmn;        // the trees of the tile's nets with >= 2 trees: mnets[mn0 .. mn0 + nmn) (tree_lane)
  int32_t tmap;            // pipelined tiles: index of the (S_H, S_V) tensor-map pair of the window's shape
                           // (one 2-D TMA copy per field), -1: the window comes by cp.async
  int32_t run0, nrun;      // noise runs[run0 .. run0 + nrun): the tile's noisy candidates in bundle order as
  int32_t nquad;           // runs of consecutive global noise indices; Philox quads they span in total
  int32_t nid0, nnoisy;    // the first run's local noise index; the tile's noisy candidates (one run: all)
};

// A run of a tile's noisy candidates (group-bundle lanes in order, padding skipped) whose global noise
// indices are consecutive: tile noise offsets [off, off + len) draw noise indices nid_base + nid ..
struct NoiseRun {
  int32_t off, len, nid, unused;   // multi-run tiles: pieces within one aligned block of 16 noise indices
};

// "General" nets (row f4'): nets with a sub-net whose candidates are not all Z(o, m)
// patterns (monotone staircases, any rectilinear path), exceed 32 candidates or come in another
// order.  They run one warp per net against global memory from explicit segment lists; their
// candidates take "virtual" slots after the bundles' (same w, m, v, p arrays).
struct GSub {
  int32_t slot;            // virtual slot of the first candidate
  int32_t n;               // candidates
  int32_t nid;             // local noise index of the first candidate, -1: a lone straight path (p = 1)
  int32_t ksub;            // kernel-order sub-net (induction outputs)
  int32_t tree;            // local tree
  int32_t gp;              // general path index of the first candidate (segment / turning-point lists)
  int32_t pad[2];
};

// Lane descriptor of a bundle slot (plan-time decode of the bundle's group structure): the lane's
// tile noise offset (bits 0-10), its group's head and end lane (11-15, 16-20) and the index of its
// sub-net within the bundle (21-25).  Padding and singleton lanes are groups of their own.
inline __host__ __device__ uint32_t lane_desc(int noff, int head, int end, int sub) {
  return (uint32_t)noff | ((uint32_t)head << 11) | ((uint32_t)end << 16) | ((uint32_t)sub << 21);
}

// A tree lane of a tile's net level: the tree (relative to the tile's first tree, bits 0-9), its net
// (offset in the tile, bits 10-20) and whether it is the net's first tree (bit 31); a net's trees
// occupy consecutive lanes of one warp.  kNoTreeLane pads.
constexpr uint32_t kNoTreeLane = 0xFFFFFFFFu;
inline __host__ __device__ uint32_t tree_lane(int tree_rel, int net_rel, bool head) {
  return (uint32_t)tree_rel | ((uint32_t)net_rel << 10) | (head ? 0x80000000u : 0u);
}

// Shared-memory offset (elements) of a pipelined tile's V field: the H field rounded up to 128 bytes
// of doubles (TMA destinations are 128-byte aligned).
inline __host__ __device__ int win_hv(int ww, int wh) { return (ww * wh + 15) & ~15; }
// Shared-memory pitch of an (even) window dimension n: n when n = 2 mod 4, else n + 2.  Lanes that
// walk across the rows of a field (one Z candidate per lane: stride = pitch) then spread over 16
// banks instead of colliding in a few (a pitch that is a multiple of 16 cells put every lane of a
// fp64 gather, or of an int32 event add, in one bank).  TMA boxes need 16-byte rows, so the pitch
// stays even.  The S window: H rows of pitch win_pitch(ww) at 0, V columns of pitch win_pitch(wh)
// at win_s_hv; the event window: three row-major fields of pitch win_pitch(ww), win_hv(pitch, wh)
// apart.
inline __host__ __device__ int win_pitch(int n) { return (n & 3) ? n : n + 2; }
inline __host__ __device__ int win_s_hv(int ww, int wh) { return win_hv(win_pitch(ww), wh); }
constexpr int kWinPad = 16;   // the S / event windows hold up to 2 (kWinMax + kWinPad) elements

struct KParams {
  // sizes
  int32_t X, Y;
  int32_t nb;               // bundles
  int32_t n_nets_l;         // local nets
  int32_t ntiles;           // pipelined tiles (persistent kernel)
  int32_t ntiles_slow;      // global / oversized tiles (one CTA each)
  int32_t XP, YP;           // even pitches of S_H rows and S_V columns
  int32_t skip;             // DGR_DEBUG_SKIP: timing knock-outs (results invalid), 0 in production
  int32_t pf;               // L2 prefetch at tile start (DGR_PF): bit 1 the trees' Adam moments (default), bit 0 also the slots' m, v, p
  int32_t ngen;             // general nets (row f4'), run by CTAs [ntiles_slow, ntiles_slow + ngen_blocks)
  int32_t ngen_blocks;
  int32_t ngsub;            // their sub-nets
  int32_t kg_h0, kg_h1, kg_v0, kg_v1;   // the rank's KG lines: H rows [kg_h0, kg_h1), V columns [kg_v0, kg_v1)
  int64_t path_base, tree_base;   // global index of the first local path / tree
  int64_t nid_base;         // global noise index of the rank's first noisy candidate
  uint64_t seed;
  uint32_t rk[20];          // Philox4x32-10 round keys of the seed (key + r (0x9E3779B9, 0xBB67AE85))
  // forest encoding
  const TileDesc* tiles;
  const TileDesc* tiles_slow;
  const int4* binfo;
  const uint32_t* pword;
  const uint32_t* ldesc;    // lane descriptors (lane_desc), per bundle slot
  const short4* sxy;        // kernel order
  const int32_t* slot_path; // local CSR path of each slot (-1 for padding); induction only
  float* wp;
  float2* mv;               // Adam moments (m, v) of each slot, interleaved (one 8-byte access)
  float* pp;                // p_i of the last forward (the reverse of that iteration reads it)
  const int32_t* net_tree_off;    // local, n_nets_l + 1
  const uint32_t* mnets;    // per tile: the trees of its nets with >= 2 trees, a lane each (tree_lane)
  const int32_t* net_gtree; // per (plan-ordered) local net: local CSR index of its first tree (tree noise key, Q7)
  int32_t perm_id;          // the plan keeps the caller's net order (plan-ordered trees = CSR trees)
  const NoiseRun* runs;     // per tile: noise runs (TileDesc run0 / nrun)
  const unsigned char* tmaps;   // CUtensorMap pairs (S_H window, S_V window), 128 B each, per window shape
  // general nets (row f4'): per net {first gtree, trees}; per tree {local tree, first gsub, sub-nets,
  // multi-tree flag}; per sub-net a GSub; per general path its segment / turning-point ranges
  const int2* gnet;
  const int4* gtree;
  const GSub* gsub;
  const int32_t* gp_seg_off;    // [n_gpath + 1] into gseg
  const int32_t* gp_tp_off;     // [n_gpath + 1] into gtp
  const short4* gseg;           // {dir, line, lo, hi}
  const short2* gtp;            // {x, y}
  long long* gdq;               // [gtrees] dq_j in 2^-32 fixed point (reverse -> net level)
  float *wt, *mt, *vt, *q;
  // grids (the exchange buffer, in this order: dH | dVT | acc)
  long long* dH;            // [Y][X] 2^-40: wire events << 16, turning points folded in (+-beta pi)
  long long* dVT;           // [X][Y] the same along columns
  long long* acc;           // [2] E[TP] and the border deficit B = sum_v VD_v (4 - deg v) of the forward
                            // in the grids (2^-24), summed by the tiles (E[WL] follows from the demand)
  const float* capH;        // [Y][X]
  const float* capVT;       // [X][Y]
  double* SH;               // [Y][XP]
  double* SVT;              // [X][YP] (contiguous after SH)
  float* dOutH;             // [Y][X]
  float* dOutVT;            // [X][Y]
  double* partial;          // [Y + X] overflow partial sums per line
  long long* lsum;          // [2] acc of the last KG's forward (KG moves acc here and clears it)
  long long* lpart;         // [Y + X] per-line sums of the demand (2^-40), for E[WL]
  double* loss;             // [4]
  double* loss_host;        // [4] or null: the caller's pinned host buffer (device alias), written by
                            // kg_loss_kernel directly instead of a copy after it (dgr_step_async)
  // induce scratch
  uint8_t* chosen;          // [n_trees_l]
  int32_t* tree_choice;     // [n_nets_l] (global tree index)
  int32_t* route;           // [n_subs_l] (global path index or -1), kernel sub-net order
  int32_t* nsize;           // [n_subs_l], kernel sub-net order
  int32_t* nucleus_tmp;     // indexed by slot: a sub-net's nucleus from its head slot on
  int32_t* DH;              // [Y][X]
  int32_t* DV;              // [Y][X]
  int32_t* VC;              // [Y][X]
  long long* iscal;         // {sum WL, sum TP}
  double* ipartial;         // [3 * nblocks]
  double* metrics;          // [5]
};

struct StepArgs {
  int64_t k;          // iteration of the reverse pass
  int64_t k_next;     // iteration of the forward pass
  float inv_t;        // 1 / temperature
  float lr_over_bc1;  // lr / (1 - beta1^(k+1))
  float inv_sqrt_bc2; // 1 / sqrt(1 - beta2^(k+1))
  float a_wl, a_via, a_of, beta, sqrt_l, f_slope;
  double beta_q;      // beta * 2^16: a turning point's pi (2^-24) -> its folded demand (2^-40)
  double beta_d, a_wl_d, via_d;   // beta, a1, a2 sqrt(L) in fp64 (the path cost's constants)
  long long beta_qi;  // the same as an integer when beta_exact
  int32_t beta_exact; // beta * 2^16 is an integer (beta a multiple of 2^-16): exact integer folds
  int32_t f_kind;
  int32_t store_d;
};

// launchers (dgr_kernels.cu)
enum TileMode { kForwardOnly = 0, kReverseForward = 1, kReverseOnly = 2 };
void launch_tiles(const KParams& p, const StepArgs& a, TileMode mode, cudaStream_t s);
void launch_kg(const KParams& p, const StepArgs& a, cudaStream_t s);
void launch_kg_loss(const KParams& p, const StepArgs& a, cudaStream_t s);   // the loss of the last KG
void launch_induce(const KParams& p, float t_final, float top_p, float beta, cudaStream_t s);
void launch_induce_metrics(const KParams& p, float beta, cudaStream_t s);
int induce_metric_blocks(const KParams& p);
size_t tile_smem_bytes();
int read_tile_prof(long long* out, int n);   // diagnostics: per-tile phase clocks
int prepare_kernels();   // sets shared-memory attributes; returns cudaError_t
int set_error(int code, const char* msg);   // the thread's dgr_last_error message (dgr_api.cu)
void clear_error();

}  // namespace dgr
