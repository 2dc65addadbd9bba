/*
 * include/tsp2opt.h -- C ABI of the B200 (sm_100a) exhaustive best-improvement
 * 2-opt library (libtsp2opt.so), after Rocki & Suda, "High Performance GPU
 * Accelerated Local Optimization in TSP", IPDPSW 2013.
 *
 * Citations "Lnn" are lines of the paper text PAPER.md (one line per page;
 * SURVEY.md §0); readings R1..R13 of garbled passages are in DESIGN.md §3.
 *
 * The operation (north_star; L12 §I.B Fig. 1-2; L14 §IV Fig. 3, Alg. 2):
 *   P[k] = coords[tour[k]] (k < n), P[n] = P[0]      (route-ordered coordinates, L18 Fig. 6)
 *   e[k] = d(P[k], P[k+1])                            (tour edges)
 *   d(a,b) = nint(sqrt((xa-xb)^2 + (ya-yb)^2))        (TSPLIB EUC_2D, exact integer; R3)
 *   for every pair 0 <= i < j <= n-1 (C(n,2) pairs; R1):
 *       delta(i,j) = d(P[i],P[j]) + d(P[i+1],P[j+1]) - e[i] - e[j]
 *   best = lowest delta, ties to the lowest Fig. 3 cell k = j(j-1)/2 + i   (R5)
 *   move = reverse tour positions i+1..j (tour[0] never moves)            (R6)
 *   local search = repeat {best; apply if delta < 0} until best delta >= 0 (R7)
 *
 * Conventions for every function:
 *   - Return TSP2OPT_OK (0) on success, a negative TSP2OPT_E* code on error,
 *     TSP2OPT_MAXITER (1) from local_search when capped.  On a validation error
 *     (EINVAL/ERANGE/ENOTPERM/ESTATE) the handle's state is unchanged.
 *   - Host pointers are only read/written during the call; the library never
 *     retains caller buffers.  All device memory is owned by the handle.
 *   - Functions are synchronous (they return after the device work finished)
 *     unless named *_async.  A handle is not thread-safe: one handle per
 *     device (and per rank); the CUDA device current at create time is used.
 *   - Coordinates are integers in [0, 2^15) (R4); 3 <= n <= 2^22 (key width, R5).
 */
#ifndef TSP2OPT_H
#define TSP2OPT_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct tsp2opt_ctx *tsp2opt_t;

enum {
    TSP2OPT_OK = 0,
    TSP2OPT_MAXITER = 1,    /* local_search applied max_iters moves and an improving move remains */
    TSP2OPT_EINVAL = -1,    /* NULL pointer, n out of range, bad rank/world, max_iters < 0, !(0<=i<j<n) */
    TSP2OPT_ERANGE = -2,    /* a coordinate outside [0, 2^15) */
    TSP2OPT_ENOTPERM = -3,  /* tour is not a permutation of 0..n-1 */
    TSP2OPT_ESTATE = -4,    /* operation needs a loaded tour (set_tour / best_move with a tour) first */
    TSP2OPT_ECUDA = -5,     /* a CUDA runtime error (message via tsp2opt_last_error) */
    TSP2OPT_ENCCL = -6,     /* an NCCL error (sharded handles) */
    TSP2OPT_ENOMEM = -7     /* device or pinned host allocation failed */
};

#define TSP2OPT_MAX_N (1 << 22)
#define TSP2OPT_COORD_LIMIT (1 << 15)
#define TSP2OPT_NCCL_ID_BYTES 128

/* Create a single-GPU handle.  coords_xy: host int32[2n] = x0,y0,x1,y1,...
 * (copied to the device once, L14 Alg. 2 step 1).  *out receives the handle. */
int tsp2opt_create(const int32_t *coords_xy, int32_t n, tsp2opt_t *out);

/* Sharded handle for one rank of `world` ranks (one GPU each, one node).
 * The triangular tile space of the sweep is split into `world` contiguous
 * ranges of equal pair count; coordinates, tour and edges are replicated; one
 * ncclAllReduce(int64, MIN) of the packed best-move key per sweep (SURVEY.md
 * §8(e); L18 §VI "dividing the 2-opt task between multiple devices").
 * nccl_id: TSP2OPT_NCCL_ID_BYTES bytes from tsp2opt_nccl_unique_id() on rank 0,
 * broadcast by the caller.  Every rank must make the same sequence of calls;
 * outputs are identical on all ranks.  world == 1 is allowed: with
 * nccl_id == NULL there is no NCCL; with an id, a one-rank communicator runs
 * the same allreduce path (the sharded code path on a single GPU). */
int tsp2opt_create_sharded(const int32_t *coords_xy, int32_t n, int32_t rank, int32_t world,
                           const void *nccl_id, tsp2opt_t *out);

/* Write an NCCL unique id (TSP2OPT_NCCL_ID_BYTES bytes) into out. */
int tsp2opt_nccl_unique_id(void *out);

/* Sharded handle whose per-sweep allreduce-min (L18
 * §VI "dividing the 2-opt task between multiple devices") runs over PEER
 * MEMORY instead of NCCL: each rank's key is stored into every other rank's
 * mailbox (CUDA IPC mapping: NVLink / NVSwitch peer memory across GPUs, the
 * same HBM for ranks sharing a GPU) and each rank takes the minimum of what
 * arrived -- one 32-thread kernel per sweep, no NCCL.  Same tiling, results
 * and call discipline as tsp2opt_create_sharded.  1 <= world <=
 * TSP2OPT_P2P_MAX_WORLD.  The handle is unusable (ESTATE) until every rank
 * has called tsp2opt_p2p_connect with all ranks' exported mailboxes.
 * A rank that stops issuing sweeps makes its peers' exchange time out after
 * about 30 s: the call returns ECUDA and the handle must be destroyed. */
#define TSP2OPT_P2P_MAX_WORLD 8
#define TSP2OPT_P2P_HANDLE_BYTES 64
int tsp2opt_create_sharded_p2p(const int32_t *coords_xy, int32_t n, int32_t rank, int32_t world, tsp2opt_t *out);

/* Export this rank's mailbox (a cudaIpcMemHandle_t, TSP2OPT_P2P_HANDLE_BYTES
 * bytes) into out; the caller all-gathers the world exports in rank order. */
int tsp2opt_p2p_export(tsp2opt_t h, void *out);

/* Map the other ranks' mailboxes: handles = world * TSP2OPT_P2P_HANDLE_BYTES
 * bytes in rank order (this rank's own entry is ignored).  EINVAL for a
 * handle not created by tsp2opt_create_sharded_p2p, ESTATE if already
 * connected, ECUDA if a mailbox cannot be mapped (nothing stays mapped). */
int tsp2opt_p2p_connect(tsp2opt_t h, const void *handles);

/* Release all device memory, streams, graphs and the NCCL communicator. */
void tsp2opt_destroy(tsp2opt_t h);

/* Use `cuda_stream` (a cudaStream_t, e.g. torch.cuda.current_stream().cuda_stream)
 * for all subsequent work; NULL selects the handle's own non-blocking stream. */
int tsp2opt_set_stream(tsp2opt_t h, void *cuda_stream);

/* Load a tour: host int32[n] permutation (validated on the host, O(n)), then
 * the route-order gather P[k] = coords[tour[k]] and the edge pass e[k] run on
 * the device (L18 Fig. 6 "array of ordered coordinates").  */
int tsp2opt_set_tour(tsp2opt_t h, const int32_t *tour);

/* Same with a DEVICE pointer (int32[n] in this GPU's memory), enqueued on the
 * handle's stream without a host sync; the permutation check runs on the device
 * and a violation surfaces as TSP2OPT_ENOTPERM from the next synchronous call
 * (tsp2opt_sync / best_move / get_tour), which also clears the loaded tour. */
int tsp2opt_set_tour_device_async(tsp2opt_t h, const int32_t *d_tour);

/* One exhaustive sweep (L14 Alg. 2 steps 2-6): if tour != NULL it is loaded
 * first (as tsp2opt_set_tour), else the current tour is used.  Returns the best
 * move (i, j, delta); at a 2-opt local minimum this is (0, 1, 0) (R7).
 * Does not modify the tour. */
int tsp2opt_best_move(tsp2opt_t h, const int32_t *tour, int32_t *i, int32_t *j, int32_t *delta);

/* Apply the 2-opt move (i, j), 0 <= i < j <= n-1: reverse positions i+1..j of
 * the tour (L12 "reversing order of sub-tour"); edges and length are updated
 * on the device.  Any valid pair is accepted (improving or not). */
int tsp2opt_apply(tsp2opt_t h, int32_t i, int32_t j);

/* Enqueue `count` device-resident iterations {sweep; [allreduce]; apply if
 * delta < 0} on the handle's stream, no host sync (the bench's timed step).
 * Iterations after convergence are no-ops.  Needs a loaded tour. */
int tsp2opt_iterate_async(tsp2opt_t h, int32_t count);

/* Wait for the handle's stream; report the device-side status:
 * *iterations = moves applied since the tour was loaded, *length = current
 * tour length, *converged = 1 at a local minimum, 2 if capped, 0 otherwise;
 * *last_i/_j/_delta = the most recent sweep's best move.  Any pointer may be NULL. */
int tsp2opt_sync(tsp2opt_t h, int64_t *iterations, int64_t *length, int32_t *converged,
                 int32_t *last_i, int32_t *last_j, int32_t *last_delta);

/* Best-improvement 2-opt local search (L12 §I.B; north_star).  tour: host
 * int32[n], in: start tour, out: tour at the local minimum (or after
 * max_iters moves).  max_iters >= 0 caps the number of applied moves
 * (TSP2OPT_MAX_ITERS_UNBOUNDED = no cap).  *length = final tour length,
 * *iterations = applied moves.  Returns TSP2OPT_OK at a local minimum,
 * TSP2OPT_MAXITER if max_iters moves were applied and an improving move remains. */
#define TSP2OPT_MAX_ITERS_UNBOUNDED INT64_MAX
/* tour == NULL: start from the handle's current tour (set_tour, mf_tour, a
 * previous search) and leave the result on the device (read it with
 * tsp2opt_get_tour); TSP2OPT_ESTATE if there is none. */
int tsp2opt_local_search(tsp2opt_t h, int32_t *tour, int64_t max_iters, int64_t *length,
                         int64_t *iterations);

/* Iterated Local Search (L10 Algorithm 1; L18 §V: random start tour, "a simple
 * doublebridge move as a perturbation technique"), device-resident:
 *   s* = local_search(tour); repeat `iterations` times:
 *     s' = double_bridge(s*, cuts(seed, t)); s*' = local_search(s');
 *     s* = s*' if length(s*') < length(s*)                  (readings R14-R16)
 * cuts: splitmix64 output 3t+k of `seed` gives segment length
 * l_k = 1 + out % max(1, (n-1)/3); a = l0, b = a + l1, c = b + l2; s' = A C B D
 * for s* = A B C D cut at a < b < c (no perturbation when n < 8).
 * tour: host int32[n], in = start tour, out = best tour; *length its length;
 * lengths (NULL or int64[iterations+1]) = best length after each step.
 * local_search is the handle's variant (set_option: pruned, first improvement,
 * 2.5-opt; oracle_ils_mode), best-improvement 2-opt by default. */
int tsp2opt_ils(tsp2opt_t h, int32_t *tour, int64_t iterations, uint64_t seed, int64_t *length,
                int64_t *lengths);

/* Batched local search of `batch` independent instances of the same size n
 * (3 <= n <= 4096), one CTA per instance, everything in shared memory
 * (the paper's small-n case, L18 §V "smaller than 200").
 * Stateless (no handle; uses the current CUDA device).  coords_xy: host
 * int32[batch * 2n] (instance b at offset 2n*b); tours: host int32[batch * n],
 * in = start tours, out = local minima (or after max_iters moves);
 * lengths / iterations: int64[batch].  Same result per instance as
 * tsp2opt_local_search.  Errors as tsp2opt_create / set_tour; nothing is
 * written on error. */
int tsp2opt_batch_local_search(const int32_t *coords_xy, int32_t n, int32_t batch, int32_t *tours,
                               int64_t max_iters, int64_t *lengths, int64_t *iterations);

/* The same on DEVICE buffers (same layouts), enqueued on `stream`
 * (cudaStream_t, NULL = legacy default stream); returns after the launch.
 * Contents are validated on the device: an instance whose tour is not a
 * permutation or whose coordinates leave [0, 2^15) gets lengths[b] =
 * iterations[b] = -1 and its tour is left unchanged.  The caller owns all
 * buffers and synchronises the stream before reading them. */
int tsp2opt_batch_local_search_async(const int32_t *d_coords_xy, int32_t n, int32_t batch, int32_t *d_tours,
                                     int64_t max_iters, int64_t *d_lengths, int64_t *d_iterations, void *stream);

/* Batched Iterated Local Search: `batch` independent replicas of L10
 * Algorithm 1 ("batched multi-replica runs for n < 200";
 * L18 §V: the paper's GPU ILS gave no speedup below 200 cities), one CTA per
 * replica, everything in shared memory (3 <= n <= 4096).  Replica b runs
 * exactly what tsp2opt_ils(h_b, tour_b, iterations, seeds[b]) runs (same
 * double-bridge cuts and acceptance, readings R14-R16) on its own instance.
 * coords_xy: host int32[batch * 2n] (replica b at offset 2n*b; repeat one
 * instance for multi-start runs); tours: host int32[batch * n], in = start
 * tours, out = best tours; seeds: uint64[batch]; lengths: int64[batch] best
 * lengths; history (or NULL): int64[batch * (iterations + 1)], the best length
 * after each step.  Errors as tsp2opt_batch_local_search; nothing is written
 * on error. */
int tsp2opt_batch_ils(const int32_t *coords_xy, int32_t n, int32_t batch, int32_t *tours, int64_t iterations,
                      const uint64_t *seeds, int64_t *lengths, int64_t *history);

/* The same on DEVICE buffers, enqueued on `stream`; an invalid replica (not a
 * permutation, coordinate out of range) gets lengths[b] = -1 and keeps its
 * tour.  The caller synchronises the stream before reading. */
int tsp2opt_batch_ils_async(const int32_t *d_coords_xy, int32_t n, int32_t batch, int32_t *d_tours,
                            int64_t iterations, const uint64_t *d_seeds, int64_t *d_lengths, int64_t *d_history,
                            void *stream);

/* Or-opt local search (SURVEY §8(f) NEXT-4 "2.5-opt/Or-opt variants"; L18 §V
 * "more sophisticated algorithms such as 3-opt, k-opt or LK"; L26 §VII; the
 * paper gives no definition: reading R21).  The
 * neighbourhood is 2-opt plus moving a segment of L = 1, 2 or 3 cities, in
 * either orientation, into another edge, over the pairs 0 <= i < j <= n-1 of
 * reading R1, 13 moves per pair:
 *   type 0: the 2-opt move (reverse positions i+1..j);
 *   type 1 + 4(L-1) + 2*dir + rev (needs j >= i+L+1): dir 0 moves
 *   t[i+1..i+L] between t[j] and t[j+1], dir 1 moves t[j-L+1..j] between
 *   t[i] and t[i+1]; rev = 1 inserts the segment reversed.
 * Best improvement: each step applies the lowest (delta, Fig. 3 cell
 * j(j-1)/2+i, type) with delta < 0; t[0] never moves.  Stateless (no handle;
 * current CUDA device, legacy default stream).  coords_xy: host int32[2n] in
 * [0, 2^15); tour: host int32[n], in = start tour, out = the Or-opt local
 * minimum (or the tour after max_iters moves); *length / *iterations (or NULL)
 * = final length and moves applied; trace_ijdt (NULL iff trace_cap == 0):
 * int32[4*trace_cap] rows (i, j, delta, type) of the first trace_cap moves.
 * 3 <= n <= TSP2OPT_OROPT_MAX_N (the key packs i and j in 20 bits).  Returns
 * TSP2OPT_OK at a local minimum, TSP2OPT_MAXITER when capped with an
 * improving move left; errors as tsp2opt_create / set_tour, or EINVAL
 * (max_iters < 0, trace_cap < 0); nothing is written on error. */
#define TSP2OPT_OROPT_MAX_N (1 << 20)
int tsp2opt_oropt_local_search(const int32_t *coords_xy, int32_t n, int32_t *tour, int64_t max_iters,
                               int64_t *length, int64_t *iterations, int32_t *trace_ijdt, int64_t trace_cap);

/* One Or-opt sweep: the best move (i, j, type, delta) of `tour` (host
 * int32[n], not modified), (0, 1, 0, 0) at a local minimum.  Arguments and
 * errors as tsp2opt_oropt_local_search. */
int tsp2opt_oropt_best_move(const int32_t *coords_xy, int32_t n, const int32_t *tour, int32_t *i, int32_t *j,
                            int32_t *type, int32_t *delta);

/* Or-opt sweep kernel selection for this process (no result depends on it;
 * DESIGN.md §5.15): filter -1 = by size (the FP32 filter from n > 2048), 0 =
 * exact walk only, 1 = FP32 filter + seeded bound; naive 1 = the one-thread-
 * per-cell kernel (filter ignored), 0 = the tiled kernel.  Overrides the
 * TSP2OPT_OROPT_FILTER / TSP2OPT_OROPT_NAIVE environment defaults.  Not
 * thread-safe against a concurrent Or-opt call.  Returns EINVAL for other
 * values. */
int tsp2opt_oropt_config(int32_t filter, int32_t naive);

/* Multiple Fragment (greedy) start tour, computed on the device (SURVEY §8(f)
 * NEXT-1; L22 §V "an initial solution based on the Multiple Fragment(Greedy)
 * heuristic[18]"; definition, tie-break and orientation: DESIGN.md R17 --
 * edges by increasing (d, min id, max id), tour starting 0 -> lower-id
 * neighbour).  It becomes the handle's current tour (local_search with
 * tour == NULL continues from it).  tour_out: host int32[n] or NULL;
 * *length (or NULL) = its length; *rounds (or NULL) = parallel rounds used.
 * The first call allocates a workspace of about (16*8 + 100) bytes per city,
 * kept until destroy.  Errors: EINVAL (h NULL), ECUDA / ENOMEM. */
int tsp2opt_mf_tour(tsp2opt_t h, int32_t *tour_out, int64_t *length, int32_t *rounds);

/* Copy the current tour (host int32[n]) and its length out. */
int tsp2opt_get_tour(tsp2opt_t h, int32_t *tour_out, int64_t *length);

/* Execution options (NEIGHBOURS, NODE_INSERTION and FIRST_IMPROVEMENT select the method; the others change
 * no result; all results stay bit-exact with the corresponding oracle):
 *  TSP2OPT_OPT_TILE_BOUNDS (default 3 from 1e8 pairs per rank, else 1): 1 = skip a tile of the sweep when the
 *      bounding boxes of its row and column cities prove that no pair can pass
 *      the per-pair necessary condition; 2 = the same, plus a
 *      pre-sweep cull (per-block boxes, one test per tile with delta < 0 as the
 *      condition) so the sweep launches over the kept tiles only; 0 tests every
 *      pair individually (the pair-check throughput the bench reports); 3 = the
 *      culled sweep made incremental: each tile keeps its own minimum over its
 *      improving pairs, and after a move only the tiles with a row or column
 *      position in the move's [i, j] are culled / re-swept, the rest keep their
 *      minimum.
 *  TSP2OPT_OPT_SEED (default 0): start each tile from its own minimum of the
 *      previous sweep when the applied move leaves that pair intact.
 *  TSP2OPT_OPT_PERSISTENT (default 2): local_search loop, 0 = one sweep and one
 *      apply kernel per iteration, 1 = one persistent cooperative launch,
 *      2 = choose by size (world == 1 only).
 *  TSP2OPT_OPT_TRACE (default 0): record the (i, j, delta) of the first `value`
 *      moves applied by iterate_async / local_search since the tour was loaded
 *      (read with tsp2opt_get_trace); 0 frees the buffer.
 *  TSP2OPT_OPT_NEIGHBOURS (default 0, at most TSP2OPT_MAX_NEIGHBOURS): K > 0
 *      switches best_move / local_search / ils of this handle to the
 *      neighbourhood-pruned 2-opt (L18 §V "limiting
 *      the neighborhood", L26 §VII "neighborhood pruning ... at the cost of the
 *      quality of the solution"; reading R18): only the moves that
 *      create an edge {a, c} with c among the K nearest cities of a by (d, id)
 *      or a among those of c; best = lowest (delta, Fig. 3 cell) over them,
 *      else (0, 1, 0).  O(nK) per sweep instead of C(n,2); the result equals
 *      oracle_pruned_best_move, not the full sweep's.  The exact candidate
 *      lists are built on the device on first use (8 * 16 * n bytes).
 *      0 restores the full neighbourhood.
 *  TSP2OPT_OPT_NODE_INSERTION (default 0): 1 switches best_move / apply /
 *      iterate_async / local_search to best-improvement 2.5-opt (SURVEY.md
 *      §8(f) NEXT-4; L26 §VII "more complex local search algorithms such as
 *      2.5-opt"; reading R19): per pair 0 <= i < j <= n-1 three
 *      moves -- type 0 the 2-opt move, type 1 (j >= i+2) city t[i+1] into the
 *      edge (t[j], t[j+1]), type 2 (j >= i+2) city t[j] into the edge
 *      (t[i], t[i+1]); best = lowest (delta, Fig. 3 cell, type), else
 *      (0, 1, 0).  best_move reports (i, j, delta) and its type is the lowest
 *      reaching delta at (i, j) (tsp2opt_best_move_typed reports it).  Type 1
 *      rotates positions i+1..j left by one, type 2 right by one; t[0] never
 *      moves.  Results equal oracle25_*.  Not with TSP2OPT_OPT_NEIGHBOURS > 0
 *      or first improvement (EINVAL); the sweep uses R = 7 rows per lane (no
 *      persistent loop).
 *  TSP2OPT_OPT_FIRST_IMPROVEMENT (default 0): 1 = first improvement (SURVEY.md
 *      §8(f) NEXT-4; reading R20): best_move returns the improving
 *      pair with the lowest Fig. 3 cell (the first one the paper's sequential
 *      pair order reaches) instead of the lowest delta, with its exact delta;
 *      local_search applies it and restarts.  With TSP2OPT_OPT_NEIGHBOURS it
 *      is the lowest improving cell of M_K (oracle_pruned_first_move).  Not
 *      with TSP2OPT_OPT_NODE_INSERTION (EINVAL).  Equals oracle_first_*.
 *  tsp2opt_ils runs its local searches with the handle's variant
 *      (oracle_ils_mode).
 * Returns TSP2OPT_EINVAL for an unknown option or value. */
#define TSP2OPT_OPT_TILE_BOUNDS 1
#define TSP2OPT_OPT_SEED 2
#define TSP2OPT_OPT_PERSISTENT 3
#define TSP2OPT_OPT_TRACE 4
#define TSP2OPT_OPT_NEIGHBOURS 5
#define TSP2OPT_MAX_NEIGHBOURS 16
#define TSP2OPT_OPT_NODE_INSERTION 6
#define TSP2OPT_OPT_FIRST_IMPROVEMENT 7
int tsp2opt_set_option(tsp2opt_t h, int32_t option, int64_t value);

/* Recorded move trace: writes min(count, cap) rows of int32 (i, j, delta) into
 * ijd (int32[3*cap]); *count = moves recorded (<= the trace capacity). */
int tsp2opt_get_trace(tsp2opt_t h, int32_t *ijd, int64_t cap, int64_t *count);

/* Diagnostics / test hooks ------------------------------------------------ */

/* 2.5-opt companions of best_move / apply / get_trace (TSP2OPT_OPT_NODE_INSERTION;
 * reading R19).  best_move_typed also reports the move type (always 0 for
 * 2-opt handles).  apply_typed applies move (i, j, type): type 0 is
 * tsp2opt_apply; types 1 and 2 need the 2.5-opt mode and 0 <= i, i+2 <= j < n
 * (else EINVAL).  get_trace_typed writes rows of int32 (i, j, delta, type)
 * into ijdt (int32[4*cap]); *count as tsp2opt_get_trace. */
int tsp2opt_best_move_typed(tsp2opt_t h, const int32_t *tour, int32_t *i, int32_t *j, int32_t *type,
                            int32_t *delta);
int tsp2opt_apply_typed(tsp2opt_t h, int32_t i, int32_t j, int32_t type);
int tsp2opt_get_trace_typed(tsp2opt_t h, int32_t *ijdt, int64_t cap, int64_t *count);

/* Restrict this handle's sweep to shard `rank` of `world` of the tile space
 * WITHOUT any collective (world = 1 restores the full sweep).  Used to check on
 * one GPU that the min over shards equals the unsharded result. */
int tsp2opt_debug_set_shard(tsp2opt_t h, int32_t rank, int32_t world);

/* Host-only planning (no GPU needed): the tile shard a handle with n cities
 * would sweep as `rank` of `world`.  *R, *warps, *tj: geometry; *ntiles,
 * *pairs: this shard's tile count and pair count.  If tiles_out != NULL it
 * receives 2 * min(*ntiles, cap) int32 (row start I0, column start J0) in
 * launch order; a tile covers rows [I0, min(I0 + 32*R*warps, n-1)) x columns
 * [J0, min(J0 + tj, n)), pairs i < j only. */
int tsp2opt_plan_shard(int32_t n, int32_t rank, int32_t world, int32_t *R, int32_t *warps, int32_t *tj,
                       int32_t *tiles_out, int64_t cap, int64_t *ntiles, int64_t *pairs);

/* Sweep geometry actually used: rows per thread R, warps per CTA, columns per
 * tile TJ, number of tiles and pairs of this handle's shard. */
int tsp2opt_get_geometry(tsp2opt_t h, int32_t *R, int32_t *warps, int32_t *tj,
                         int64_t *tiles, int64_t *pairs);

/* Exhaustive device self-test of the sweep kernel's arithmetic (same inline
 * device functions): (a) the exact distance d(s) over every s in [0, 2*32767^2]
 * against m^2 - m < s <= m^2 + m; (b) the squared-distance prefilter never
 * rejects: for every (dx, dy) in [0, 32767]^2 the float s(dx,dy) passes the
 * float threshold built from t = d(dx,dy).  Writes the violation counts and
 * (may be NULL) the smallest violating s and (dx << 15 | dy), or -1. */
int tsp2opt_selftest(int64_t *dist_violations, int64_t *filter_violations, int64_t *first_bad_s,
                     int64_t *first_bad_dxdy);

/* Sweep-kernel timing: enable != 0 starts recording a CUDA event pair around
 * every sweep launch of this handle (previous records are dropped); enable == 0
 * stops.  tsp2opt_profile_read waits for the stream and returns the summed
 * device time (ms) of the recorded sweep launches and their number. */
int tsp2opt_profile(tsp2opt_t h, int32_t enable);
int tsp2opt_profile_read(tsp2opt_t h, double *total_ms, int64_t *launches);

/* Exhaustive bound of the sweep's sqrt-sum prefilter input: the max relative
 * error of the kernel's MUFU.SQRT over every float in [1, 2^31] (*max_rel_err)
 * and whether sqrt(0) == 0 (*zero_ok).  DESIGN.md §5.2 needs <= 2^-21. */
int tsp2opt_selftest_sqrt(double *max_rel_err, int32_t *zero_ok);

/* Sweep counters of an instrumented build (-DTSP2OPT_STATS): out4[0] warp column
 * steps, [1] steps that took the exact path, [2] candidate pairs evaluated
 * exactly, [3] warp tiles walked (not skipped by the tile bound); -1 in
 * product builds.  reset != 0 zeroes them afterwards. */
int tsp2opt_debug_stats(int64_t *out4, int32_t reset);

/* Phase clocks of the persistent incremental local search in an instrumented
 * build (-DTSP2OPT_PHASE_TIMING), summed over iterations: out16[k] = SM clock
 * cycles CTA 0 spent in [0] dirty boxes, [1] barrier, [2] cull + kept-tile
 * sweeps, [6] clean-minimum scan, [3] barrier, [4] apply, [5] barrier; over
 * all warps, per iteration: [8] the longest cull + sweep, [9] the most kept
 * tiles of one warp, [10] the longest cull alone, [11] the kept tiles; -1 in
 * product builds.  reset != 0 zeroes them afterwards. */
int tsp2opt_debug_phases(int64_t *out16, int32_t reset);

/* Number of this library's kernel launches since load (for gpu_launches). */
int64_t tsp2opt_launch_count(void);

/* Human-readable message for a return code; last CUDA/NCCL error text. */
const char *tsp2opt_strerror(int code);
const char *tsp2opt_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* TSP2OPT_H */
