// tsp2opt_internal.h -- host-side declarations shared by the kernels and the
// C-ABI runtime of libtsp2opt.so (not part of the public ABI; see include/tsp2opt.h).
#pragma once

#include <atomic>
#include <algorithm>
#include <cstdint>
#include <cuda_runtime.h>

#include "tsp2opt_device.cuh"

namespace tsp2opt {

constexpr int kRowsLarge = 15;  // R for large n: 16 row cities per lane (8 packed FP32x2 pairs)
constexpr int kRowsSmall = 7;   // R for small / medium n
constexpr int kRows = kRowsLarge;  // the largest R (padding)
constexpr int kMaxTJ = 1024;  // columns per tile, upper bound (shared memory sizing)
constexpr int kMaxWarps = 4;  // warps per CTA, upper bound (__launch_bounds__(128))
constexpr int kPad = 32 * kRows * kMaxWarps + kMaxTJ + 8;  // P/E/tour padding beyond n

struct Geometry {
    int rows;   // R
    int warps;  // warps per CTA
    int tj;     // columns per tile
    int ti() const { return 32 * rows * warps; }
};

long long launch_count();
void count_launch(int k = 1);

// Launch with the programmatic-dependent-launch attribute (TSP2OPT_PDL=0 turns
// it off: plain stream order).  DESIGN.md §5.3.
bool pdl_enabled();
template <typename... KArgs, typename... Args>
inline cudaError_t launch_kernel_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                                     Args... args)
{
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = pdl_enabled() ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, kernel, static_cast<KArgs>(args)...);
}
constexpr int kBatchMaxN = 4096;  // batched local search: one instance per CTA, all in shared memory
size_t batch_smem_bytes(int n);
cudaError_t launch_batch_local_search(const int* coords, int* tours, int n, int batch, long long max_iters,
                                      long long* lengths, long long* iters, cudaStream_t st);
cudaError_t launch_batch_ils(const int* coords, int* tours, int n, int batch, long long iterations,
                             const unsigned long long* seeds, long long* lengths, long long* history, cudaStream_t st);
// Multiple Fragment start tour (tsp2opt_mf.cu)
constexpr int kMfK = 16;        // exact nearest neighbours kept per city
constexpr int kMfCtr = 4;       // per-round counters, x2 parities: ends, scans, accepted, pad
constexpr int kMfEdges = 8;     // kept edges so far
constexpr int kMfEndCnt = 9;    // path ends found by the closing step
constexpr int kMfEnd0 = 10;     // [2] the path's two ends
constexpr int kMfCtrInts = 16;
size_t mf_workspace_bytes(int n);
cudaError_t launch_mf_tour(const int* coords, int n, void* ws, int* tour_out, int* rounds_out, cudaStream_t st);
// Exact kMfK nearest neighbours of every city, keys (d << 22 | c) ascending by (d, c), ~0 pad
cudaError_t launch_knn(const int* coords, int n, unsigned long long* knn, cudaStream_t st);
// Neighbourhood-pruned sweep (tsp2opt_pruned.cu; reading R18): candidates of positions [p0, p1)
constexpr int kMaxNeighbours = kMfK;
cudaError_t launch_pruned_sweep(const float2* P, const int* E, const int* tour, const int* pos,
                                const unsigned long long* knn, int K, int n, int p0, int p1, Slot* slot,
                                int respect_done, int first, cudaStream_t st);
cudaError_t launch_pos(const int* tour, int* pos, int n, cudaStream_t st);
// 2.5-opt (tsp2opt_sweep25.cu; reading R19): sweep over the dense tiling with R = kRowsSmall,
// per-position removal gains G, cooperative apply resolving the move type.
size_t sweep25_smem_bytes(const Geometry& g);
cudaError_t sweep25_prepare();
cudaError_t launch_sweep25(const Geometry& g, const float2* P, const int* E, const int* G, int n, const int2* tiles,
                           int ntiles, Slot* slot, int respect_done, int flags, cudaStream_t st);
cudaError_t launch_gain(const float2* P, int* G, int n, int lo, int hi, cudaStream_t st);
int sweep25_list_grid(const Geometry& g, int ntiles);
cudaError_t launch_sweep25_list(const Geometry& g, const float2* P, const int* E, const int* G, int n,
                                const int4* list, int grid, Slot* slot, int respect_done,
                                unsigned long long* tilebest, int flags, cudaStream_t st);
cudaError_t launch_decide25(const float2* P, const int* E, const int* G, Slot* slot, cudaStream_t st);
cudaError_t launch_apply25(float2* P, int* E, int* G, int* tour, int n, const Slot* in, Slot* out,
                           long long max_moves, int explicit_move, int ei, int ej, int etype,
                           unsigned long long* trace, int* ttype, long long trace_cap, unsigned* bar, cudaStream_t st);
// Or-opt (tsp2opt_oropt.cu; reading R21): route-ordered int2 Q[n + 5], dense sweep, span apply.
// Device state of the Or-opt loop, u64 words: [0] the sweep's key, then these.
constexpr int kOrLength = 1;  // tour length (int64)
constexpr int kOrMoves = 2;   // moves applied
constexpr int kOrDone = 3;    // 0 running, 1 local minimum, 2 capped with an improving move left
constexpr int kOrCap = 4;     // max_iters
constexpr int kOrMove = 5;    // the key of the move the current iteration applies, 0 if none
constexpr int kOrSlotWords = 8;
size_t oropt_q_entries(int n);
cudaError_t launch_or_load(const int* coords, const int* tour, int2* Q, int n, unsigned long long* len, cudaStream_t st);
size_t oropt_const_entries(int n);
void or_config(int filter, int naive);
cudaError_t launch_or_sweep(const int2* Q, int4* CR, int4* CC, int n, unsigned long long* slot, cudaStream_t st);
// decide (device: done / capped / record the move) + span + commit, all reading the slot
cudaError_t launch_or_apply(const int* coords, int* tour, int2* Q, int* span, int n, unsigned long long* slot,
                            int* trace, long long trace_cap, cudaStream_t st);
void or_unpack(unsigned long long key, int* i, int* j, int* type, int* delta);
size_t sweep_smem_bytes(const Geometry& g);
cudaError_t sweep_prepare();
cudaError_t launch_load_tour(const int* coords, const int* tour_src, int* tour_dst, float2* P, int* E, int n,
                             Slot* slot, unsigned* stamp, unsigned epoch, cudaStream_t st);
cudaError_t launch_reset_key(Slot* slot, cudaStream_t st);
// P / E non-null: re-evaluate every tile minimum's positions on the new tour (else: surviving pairs only)
cudaError_t launch_global_seed(const unsigned long long* tilebest, int ntiles, Slot* slot, const float2* P,
                               const int* E, cudaStream_t st);
cudaError_t launch_first_fix(const float2* P, const int* E, Slot* slot, int respect_done, cudaStream_t st);
cudaError_t launch_double_bridge(const int* in, int* out, int n, int a, int b, int c, cudaStream_t st);
cudaError_t launch_sweep(const Geometry& g, const float2* P, const int* E, int n, const int2* tiles, int ntiles,
                         Slot* slot, int respect_done, unsigned long long* tilebest, int flags, cudaStream_t st);
// Culled sweep (TSP2OPT_OPT_TILE_BOUNDS = 2): per-block boxes, the tile cull
// into list / slot->ncull, then the sweep over the list with `grid` CTAs.
int sweep_list_grid(const Geometry& g, int ntiles);
// box + cull only (the 2.5-opt list sweep follows); G != NULL adds the gain term to the cull
cudaError_t launch_box_cull(const Geometry& g, const float2* P, const int* E, const int* G, int n, const int2* tiles,
                            int ntiles, Box* rbox, Box* cbox, int4* list, Slot* slot, int respect_done,
                            unsigned long long* tilebest, int flags, cudaStream_t st);
cudaError_t launch_cull_sweep(const Geometry& g, const float2* P, const int* E, int n, const int2* tiles,
                              int ntiles, int grid, Box* rbox, Box* cbox, int4* list, Slot* slot, int respect_done,
                              unsigned long long* tilebest, int flags, cudaStream_t st);
// Fused incremental culled sweep (after the first iteration of a TILE_BOUNDS = 3 search):
// dirty tiles enumerated from the last move via tmap, boxes recomputed in place, cull and sweep
// in one launch of `grid` one-warp CTAs (inc_sweep_grid), clean minima folded into the key.
int inc_sweep_grid(const Geometry& g);
// Persistent dense local search with dynamic warp-level tile claims (one cooperative launch).
cudaError_t launch_dense_ls(const Geometry& g, float2* P, int* E, int* tour, int n, const int2* tiles, int ntiles,
                            Slot* slots, int parity, long long max_moves, long long budget, unsigned* bar, int* ctl,
                            int flags, unsigned long long* tilebest, unsigned long long* trace, long long trace_cap,
                            cudaStream_t st);
// Persistent incremental local search (one cooperative launch, one CTA of 16 warps per SM):
// up to `budget` iterations of {dirty boxes; clean minima + cull + kept-tile sweeps; apply};
// full = 1 makes the first iteration the full culled sweep.  ctl[0] = the final slot parity.
cudaError_t launch_inc_ls(const Geometry& g, float2* P, int* E, int* tour, int n, const int2* tiles, int ntiles,
                          const int* tmap, Box* rbox, Box* cbox, Slot* slots, int parity, long long max_moves,
                          long long budget, int full, unsigned* bar, int* ctl, unsigned long long* tilebest, int flags,
                          unsigned long long* trace, long long trace_cap, int part_cols, cudaStream_t st);
// Same search with two grid barriers per move (inc_ls2_kernel): the move is applied out of place into
// P1 / E1 / T1 (np entries each, alternating with P / E / tour), and the next sweep's boxes and clean
// minima are computed in the same phase.  ws: inc_ls2_ws_bytes (the barrier counter, the dense tile
// minima and their group minima; the minima initialised to all-ones once).  part_cols: columns per
// part of a kept tile (0: the default); part_bound: the tile bound on every part.  P / E / tour hold the
// current state when it returns.
size_t inc_ls2_ws_bytes(const Geometry& g, int n);
cudaError_t launch_inc_ls2(const Geometry& g, float2* P, int* E, int* tour, float2* P1, int* E1, int* T1, int n,
                           int np, const int* tmap, Box* rbox, Box* cbox, void* ws, Slot* slots, int parity,
                           long long max_moves, long long budget, int full, int* ctl, int flags,
                           unsigned long long* trace, long long trace_cap, int part_cols, int part_bound,
                           cudaStream_t st);
// One grid barrier per move (inc_ls1_kernel): the dirty tiles of move m are swept in the same phase as
// its out-of-place apply, reading the pre-move buffers through the mirror map, with conservative boxes
// for the cull.  ws: inc_ls1_ws_bytes (barrier counter, keys, dense tile and group minima, two box
// buffers; all-ones once, so that the minima of tiles that do not exist read as none).  Every launch starts with a full sweep; the slot comes back with
// seed_ok = 0.
size_t inc_ls1_ws_bytes(const Geometry& g, int n);
cudaError_t launch_inc_ls1(const Geometry& g, float2* P, int* E, int* tour, float2* P1, int* E1, int* T1, int n,
                           int np, const int* tmap, void* ws, Slot* slots, int parity, long long max_moves,
                           long long budget, int* ctl, int flags, unsigned long long* trace, long long trace_cap,
                           int part_cols, cudaStream_t st);
cudaError_t launch_inc_sweep(const Geometry& g, const float2* P, const int* E, int n, const int2* tiles, int ntiles,
                             const int* tmap, int grid, Box* rbox, Box* cbox, Slot* slot, int respect_done,
                             unsigned long long* tilebest, int flags, cudaStream_t st);
cudaError_t launch_apply(float2* P, int* E, int* tour, int n, const Slot* in, Slot* out, long long max_moves,
                         int explicit_move, int ei, int ej, unsigned long long* trace, long long trace_cap,
                         int* pos, cudaStream_t st);
cudaError_t launch_local_search(const Geometry& g, float2* P, int* E, int* tour, int n, const int2* tiles, int ntiles,
                                Slot* slots, int parity, long long max_moves, long long budget, unsigned* bar,
                                int* ctl, unsigned long long* tilebest, int flags, unsigned long long* trace,
                                long long trace_cap, cudaStream_t st);
// Allreduce-min of the slot key over peer-memory mailboxes (tsp2opt_p2p.cu): peers[r] = rank r's
// mailbox mapped into this process (peers[rank] = the own one).
cudaError_t launch_p2p_min(Slot* slot, Mailbox* const* peers, int rank, int world, int respect_done,
                           cudaStream_t st);
cudaError_t read_stats(long long* out4, int reset);
cudaError_t read_phases(long long* out16, int reset);
cudaError_t run_selftest_sqrt(double* max_rel, int* zero_ok);
cudaError_t run_selftest(long long* out4);  // dist_bad, filter_bad, first bad s, first bad dx<<15|dy

}  // namespace tsp2opt
