// tsp2opt_api.cu -- C ABI (include/tsp2opt.h) and host runtime of libtsp2opt.so.
//
// Owns the device state of one instance (one GPU, one rank): coordinates,
// tour, route-ordered coordinates P, edges E, the ping-pong Slot pair, the
// sweep's tile table; drives the kernels of tsp2opt_kernels.cu on one stream;
// for sharded handles owns an NCCL communicator and performs one 8-byte
// ncclAllReduce(MIN) of the packed best-move key per sweep.
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include <nccl.h>

#include "../../include/tsp2opt.h"
#include "tsp2opt_internal.h"

using namespace tsp2opt;
static_assert(kMaxNeighbours == TSP2OPT_MAX_NEIGHBOURS, "candidate list width");

namespace {

thread_local std::string g_last_error;

int cuda_fail(cudaError_t e, const char* what)
{
    g_last_error = std::string(what) + ": " + cudaGetErrorString(e);
    return e == cudaErrorMemoryAllocation ? TSP2OPT_ENOMEM : TSP2OPT_ECUDA;
}
int nccl_fail(ncclResult_t r, const char* what)
{
    g_last_error = std::string(what) + ": " + ncclGetErrorString(r);
    return TSP2OPT_ENCCL;
}

#define CUDA_TRY(call)                                   \
    do {                                                 \
        cudaError_t e_ = (call);                         \
        if (e_ != cudaSuccess) return cuda_fail(e_, #call); \
    } while (0)

struct Tile {
    int i0, j0;
    long long pairs;
};

}  // namespace

struct tsp2opt_ctx {
    int n = 0;
    int rank = 0, world = 1;          // NCCL sharding
    int shard_rank = 0, shard_world = 1;  // tile range actually swept (== rank/world unless debug)
    int device = 0;
    cudaStream_t own_stream = nullptr;
    cudaStream_t stream = nullptr;
    int* d_coords = nullptr;    // int32[2n]
    int* d_tour = nullptr;      // int32[n + pad]
    int* d_tour_in = nullptr;   // int32[n] staging for host tours
    float2* d_P = nullptr;      // [n + 1 + pad] biased route-ordered coordinates
    int* d_E = nullptr;         // [n + pad] edges
    float2* d_P_alt = nullptr;  // alternate P / E / tour of the two-barrier persistent search (allocated on first use)
    int* d_E_alt = nullptr;
    int* d_tour_alt = nullptr;
    void* d_inc2_ws = nullptr; // its barrier counter, dense tile minima and group minima (inc_ls2_ws_bytes)
    Geometry igeo{};            // its culled tiling (own tile map and boxes)
    int* d_itmap = nullptr;
    Box* d_irbox = nullptr;
    Box* d_icbox = nullptr;
    int inc_barriers = 1;       // TSP2OPT_INC_BARRIERS=2: two grid barriers per move (inc_ls2_kernel); 3: the
                                // three-barrier kernel (in-place apply)
    void* d_inc1_ws = nullptr;  // inc_ls1_kernel workspace (inc_ls1_ws_bytes), allocated with the inc2 one
    int inc_part = -1;          // TSP2OPT_INC_PART: columns per part of a kept tile (-1: the default; 0 with the
                                // three-barrier kernel: one warp per whole tile)
    int inc_part_bound = 0;     // TSP2OPT_INC_PART_BOUND=1: the tile bound on every part (measured 4 % slower)
    // Automatic switch of the dense best-improvement loop (TILE_BOUNDS 1, n ~ 7e3) to the persistent
    // incremental search once the tour is spatially coherent: length < kAutoIncRho * sqrt(n * A),
    // A = the coordinates' bounding-box area (a random tour is ~0.5 sqrt(n) times that, a good one
    // ~0.75-1).  Off when TILE_BOUNDS is set by option or environment (TSP2OPT_AUTO_INC=0: off).
    bool auto_inc = false;
    double rho_unit = 0.0;      // sqrt(n * A)
    Slot* d_slots = nullptr;    // [2]
    unsigned* d_stamp = nullptr;  // [n] permutation check
    unsigned* d_bar = nullptr;    // [2] grid barrier of the persistent local search (count, generation)
    int* d_ctl = nullptr;         // [1] parity the persistent local search ended on
    int* h_ctl = nullptr;         // pinned readback of d_ctl
    int persistent = 2;           // local_search loop: 0 per-iteration kernels, 1 persistent launch, 2 auto
    int2* d_tiles = nullptr;    // this shard's tiles
    unsigned long long* d_tilebest = nullptr;  // [ntiles] per-tile minima of the last sweep (next seed)
    bool seed_next = false;     // seed each tile with its surviving minimum of the previous sweep (TSP2OPT_SEED=1;
                                // measured neutral-to-slower at n = 1002 .. 33810, so off by default)
    int tile_bounds = 1;        // TSP2OPT_OPT_TILE_BOUNDS: 0 off, 1 per-tile bound inside the sweep, 2 also the
                                // pre-sweep cull (box + cull kernels; the sweep runs over the kept tiles only)
    Box* d_rbox = nullptr;      // culled sweep: per row-block / column-chunk summaries
    Box* d_cbox = nullptr;
    // The culled sweep has its own tiling (narrower column chunks: a finer cull
    // and more, shorter work items for the few tiles a coherent tour keeps).
    Geometry cgeo{};
    std::vector<Tile> all_ctiles;
    int2* d_ctiles = nullptr;   // this shard's cull tiles
    unsigned long long* d_ctilebest = nullptr;  // their per-tile minima (seeds)
    int4* d_list = nullptr;     // kept cull tiles (I0, J0, index) [nctiles]
    int* d_tmap = nullptr;      // [nrb * ncc] (row block, column chunk) -> this shard's cull-tile index, -1 if none
    int inc_grid = 0;           // one-warp CTAs of the fused incremental sweep (co-resident)
    bool inc_fused = true;      // TSP2OPT_INC_FUSED=0: the box + cull + list kernels on every iteration
    bool inc_persistent = true; // TSP2OPT_INC_PERSISTENT=0: per-iteration launches instead of one cooperative launch
    bool dense_ls = false;      // TSP2OPT_DENSE_LS=1: the persistent dense loop with dynamic claims above the round-robin
                                // persistent size (measured slower at C3: 30-38 vs 22 us per move, r02_exp_dense_ls.jsonl)
    int nctiles = 0;
    int list_grid = 0;          // CTAs of the culled sweep (co-resident)
    int list25_grid = 0;        // CTAs of the 2.5-opt culled sweep
    int last_tiling = -1;       // tiling of the previous sweep (0 dense, 1 cull): seeds are per tiling
    bool inc_valid = false;     // the stored per-tile minima are those of an incremental sweep of the current tiling
    int global_seed = 0;        // TSP2OPT_GLOBAL_SEED=1: dense sweeps start from the best surviving tile minimum
                                // (2: from every tile minimum's positions re-evaluated on the new tour)
                                // (measured: C4 random 8 % faster, C2 / C3 2-10 % slower; profiles/r01_global_seed.jsonl)
    unsigned long long* d_trace = nullptr;  // [trace_cap] keys of the applied moves (TSP2OPT_OPT_TRACE)
    int* d_best = nullptr;      // [n] best tour of an ILS run
    void* d_mf_ws = nullptr;    // Multiple Fragment workspace (mf_workspace_bytes), allocated on first use
    int mf_rounds = 0;          // rounds of the last tsp2opt_mf_tour
    int nbr_k = 0;              // TSP2OPT_OPT_NEIGHBOURS: 0 full neighbourhood, K > 0 the pruned M_K (reading R18)
    unsigned long long* d_knn = nullptr;  // [n * kMaxNeighbours] exact nearest-neighbour keys (d << 22 | c)
    int* d_pos = nullptr;       // [n] inverse permutation pos[tour[k]] = k (pruned sweep only)
    int or25 = 0;               // TSP2OPT_OPT_NODE_INSERTION: 1 = 2.5-opt (2-opt plus node insertion, reading R19)
    int first = 0;              // TSP2OPT_OPT_FIRST_IMPROVEMENT: 1 = lowest improving cell (reading R20)
    int* d_G = nullptr;         // [n + 1 + pad] removal gains g_k (2.5-opt only)
    unsigned* d_bar25 = nullptr;  // [2] grid barrier of the 2.5-opt apply
    int* d_ttype = nullptr;     // [trace_cap] move types of the traced moves (2.5-opt)
    long long trace_cap = 0;
    Slot* h_slot = nullptr;     // pinned readback
    unsigned epoch = 0;
    int parity = 0;             // iteration t reads slot[parity]
    bool has_tour = false;
    Geometry geo{};
    std::vector<Tile> all_tiles;  // sorted, all shards
    int ntiles = 0;               // tiles of this shard
    long long shard_pairs = 0;
    ncclComm_t comm = nullptr;
    // peer-memory exchange (tsp2opt_create_sharded_p2p): own mailbox, the peers' mapped ones
    bool p2p = false;
    bool p2p_ready = false;
    Mailbox* d_mbox = nullptr;
    Mailbox** d_peers = nullptr;           // [world] device array of mailbox pointers (own at [rank])
    std::vector<void*> p2p_opened;         // peers' mailboxes opened with cudaIpcOpenMemHandle
    bool profiling = false;
    std::vector<cudaEvent_t> ev_pool;  // pairs (start, stop) of recorded sweep launches
    size_t ev_used = 0;
};

namespace {

Geometry choose_geometry(long long pairs_per_rank)
{
    // Measured on B200 (tools/exp_geometry*.py): one-warp CTAs
    // and many small tiles win at every size (no intra-CTA barrier skew, the
    // hardware scheduler balances); R = 15 from ~1e8 pairs (n = 33810: local
    // search 0.63 s vs 0.68 s with R = 7), R = 7 below; columns per tile grow
    // with the pair count (n = 85900: TJ = 128 -> 0.79 ms/sweep, 60k tiles;
    // n = 7397: TJ = 16; n = 1002: TJ = 8).
    const long long p = pairs_per_rank;
    int R = p >= 100000000LL ? kRowsLarge : kRowsSmall;
    // (beyond the measured range the tile count is capped near 1e6-1e7 so the
    // host-side tile table stays small: n = 2^22 -> 18M tiles of 480 x 1024)
    int tj = p >= 100000000000LL ? 1024
             : p >= 10000000000LL ? 512
             : p >= 1000000000LL  ? 128
             : p >= 100000000LL   ? 64
             : p >= 5000000LL     ? 16
                                  : 8;
    int w = 1;
    if (const char* er = getenv("TSP2OPT_ROWS")) R = atoi(er) == kRowsSmall ? kRowsSmall : kRowsLarge;
    const char* ew = getenv("TSP2OPT_WARPS");
    const char* et = getenv("TSP2OPT_TJ");
    if (ew && et && atoi(ew) >= 1 && atoi(ew) <= kMaxWarps && atoi(et) >= 2 && atoi(et) <= kMaxTJ) {
        w = atoi(ew);
        tj = atoi(et);
    }
    return Geometry{R, w, tj};
}

// Tiles over the upper triangle only (L20 Fig. 8 "Skip unnecessary computation"):
// row blocks [I0, I0+TI) with I0 <= n-2, column chunks [J0, J0+TJ) containing a
// column j > I0; pairs = #{(i, j): I0 <= i < min(I0+TI, n-1), J0 <= j < min(J0+TJ, n), i < j}.
std::vector<Tile> build_tiles(int n, const Geometry& g)
{
    std::vector<Tile> t;
    const int TI = g.ti(), TJ = g.tj;
    for (int I0 = 0; I0 <= n - 2; I0 += TI) {
        const int rows = std::min(I0 + TI, n - 1) - I0;
        for (int J0 = ((I0 + 1) / TJ) * TJ; J0 < n; J0 += TJ) {
            const int J1 = std::min(J0 + TJ, n);
            // sum over j in [J0, J1) of min(max(j - I0, 0), rows), in closed form
            auto tri = [](long long m) { return m > 0 ? m * (m + 1) / 2 : 0; };  // 1 + 2 + ... + m
            const long long a = std::max<long long>(J0, I0), b = std::min<long long>(J1, (long long)I0 + rows);
            long long p = a < b ? tri(b - 1 - I0) - tri(a - 1 - I0) : 0;      // ramp part j - I0
            p += (long long)rows * std::max<long long>(0, J1 - std::max<long long>(J0, (long long)I0 + rows));
            if (p > 0) t.push_back({I0, J0, p});
        }
    }
    std::stable_sort(t.begin(), t.end(), [](const Tile& a, const Tile& b) { return a.pairs > b.pairs; });
    return t;
}

// Greedy LPT split of the (size-sorted) tile list into `world` shards of equal
// pair count; each shard keeps the largest-first order.
std::vector<Tile> shard_tiles(const std::vector<Tile>& all, int rank, int world, long long* pairs)
{
    std::vector<long long> load(world, 0);
    std::vector<Tile> mine;
    for (const Tile& t : all) {
        int r = (int)(std::min_element(load.begin(), load.end()) - load.begin());
        load[r] += t.pairs;
        if (r == rank) mine.push_back(t);
    }
    *pairs = load[rank];
    return mine;
}

// Upload this rank's share of one tiling: tile origins and per-tile seeds.
int upload_tiling(const std::vector<Tile>& all, int rank, int world, int2** d_tiles,
                  unsigned long long** d_best, int* ntiles, long long* pairs)
{
    std::vector<Tile> mine = shard_tiles(all, rank, world, pairs);
    std::vector<int2> host(mine.size());
    for (size_t k = 0; k < mine.size(); k++) host[k] = make_int2(mine[k].i0, mine[k].j0);
    cudaFree(*d_tiles);
    cudaFree(*d_best);
    *d_tiles = nullptr;
    *d_best = nullptr;
    if (!host.empty()) {
        CUDA_TRY(cudaMalloc(d_tiles, host.size() * sizeof(int2)));
        CUDA_TRY(cudaMalloc(d_best, host.size() * sizeof(unsigned long long)));
        CUDA_TRY(cudaMemset(*d_best, 0xFF, host.size() * sizeof(unsigned long long)));  // kKeyNone
        CUDA_TRY(cudaMemcpy(*d_tiles, host.data(), host.size() * sizeof(int2), cudaMemcpyHostToDevice));
    }
    *ntiles = (int)host.size();
    return TSP2OPT_OK;
}

int upload_shard(tsp2opt_ctx* h, int rank, int world)
{
    long long pairs = 0, cpairs = 0;
    int rc = upload_tiling(h->all_tiles, rank, world, &h->d_tiles, &h->d_tilebest, &h->ntiles, &pairs);
    if (rc) return rc;
    rc = upload_tiling(h->all_ctiles, rank, world, &h->d_ctiles, &h->d_ctilebest, &h->nctiles, &cpairs);
    if (rc) return rc;
    cudaFree(h->d_list);
    h->d_list = nullptr;
    if (h->nctiles > 0) CUDA_TRY(cudaMalloc(&h->d_list, sizeof(int4) * (size_t)h->nctiles));
    {  // (row block, column chunk) -> index in this shard's cull-tile array (the fused incremental sweep)
        const int TI = h->cgeo.ti(), TJ = h->cgeo.tj;
        const int nrb = (h->n - 1 + TI - 1) / TI, ncc = (h->n + TJ - 1) / TJ;
        std::vector<int> map((size_t)nrb * ncc, -1);
        long long unused = 0;
        std::vector<Tile> mine = shard_tiles(h->all_ctiles, rank, world, &unused);
        for (size_t k = 0; k < mine.size(); k++) map[(size_t)(mine[k].i0 / TI) * ncc + mine[k].j0 / TJ] = (int)k;
        cudaFree(h->d_tmap);
        h->d_tmap = nullptr;
        CUDA_TRY(cudaMalloc(&h->d_tmap, sizeof(int) * map.size()));
        CUDA_TRY(cudaMemcpy(h->d_tmap, map.data(), sizeof(int) * map.size(), cudaMemcpyHostToDevice));
        h->inc_grid = inc_sweep_grid(h->cgeo);
    }
    h->list_grid = sweep_list_grid(h->cgeo, h->nctiles);
    if (const char* el = getenv("TSP2OPT_LIST_GRID"))  // experiment: cap the list sweep's co-resident grid
        if (atoi(el) > 0) h->list_grid = std::min(h->list_grid, atoi(el));
    h->list25_grid = sweep25_list_grid(h->cgeo, h->nctiles);
    h->last_tiling = -1;
    h->inc_valid = false;
    h->shard_pairs = pairs;
    h->shard_rank = rank;
    h->shard_world = world;
    return TSP2OPT_OK;
}

void free_ctx(tsp2opt_ctx* h)
{
    if (!h) return;
    if (h->comm) ncclCommDestroy(h->comm);
    cudaFree(h->d_coords);
    cudaFree(h->d_tour);
    cudaFree(h->d_tour_in);
    cudaFree(h->d_P);
    cudaFree(h->d_E);
    cudaFree(h->d_P_alt);
    cudaFree(h->d_E_alt);
    cudaFree(h->d_tour_alt);
    cudaFree(h->d_inc2_ws);
    cudaFree(h->d_inc1_ws);
    cudaFree(h->d_itmap);
    cudaFree(h->d_irbox);
    cudaFree(h->d_icbox);
    cudaFree(h->d_slots);
    cudaFree(h->d_stamp);
    cudaFree(h->d_bar);
    cudaFree(h->d_ctl);
    if (h->h_ctl) cudaFreeHost(h->h_ctl);
    cudaFree(h->d_tiles);
    cudaFree(h->d_tilebest);
    cudaFree(h->d_ctiles);
    cudaFree(h->d_ctilebest);
    cudaFree(h->d_list);
    cudaFree(h->d_tmap);
    for (void* p : h->p2p_opened)
        if (p) cudaIpcCloseMemHandle(p);
    cudaFree(h->d_peers);
    cudaFree(h->d_mbox);
    cudaFree(h->d_rbox);
    cudaFree(h->d_cbox);
    cudaFree(h->d_trace);
    cudaFree(h->d_best);
    cudaFree(h->d_mf_ws);
    cudaFree(h->d_knn);
    cudaFree(h->d_pos);
    cudaFree(h->d_G);
    cudaFree(h->d_bar25);
    cudaFree(h->d_ttype);
    if (h->h_slot) cudaFreeHost(h->h_slot);
    for (cudaEvent_t e : h->ev_pool) cudaEventDestroy(e);
    if (h->own_stream) cudaStreamDestroy(h->own_stream);
    delete h;
}

int validate_coords(const int32_t* xy, int32_t n)
{
    if (!xy) return TSP2OPT_EINVAL;
    if (n < 3 || n > TSP2OPT_MAX_N) return TSP2OPT_EINVAL;
    for (long long k = 0; k < 2LL * n; k++)
        if (xy[k] < 0 || xy[k] >= TSP2OPT_COORD_LIMIT) return TSP2OPT_ERANGE;
    return TSP2OPT_OK;
}

int validate_tour(const int32_t* t, int n)
{
    if (!t) return TSP2OPT_EINVAL;
    std::vector<unsigned char> seen(n, 0);  // bytes: the check stays in the host's L2
    for (int k = 0; k < n; k++) {
        if (t[k] < 0 || t[k] >= n || seen[t[k]]) return TSP2OPT_ENOTPERM;
        seen[t[k]] = 1;
    }
    return TSP2OPT_OK;
}

int read_slot(tsp2opt_ctx* h)
{
    CUDA_TRY(cudaMemcpyAsync(h->h_slot, h->d_slots + h->parity, sizeof(Slot), cudaMemcpyDeviceToHost, h->stream));
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    if (h->h_slot->done & kDoneExchangeTimeout) {
        g_last_error = "peer-memory exchange timed out (a rank stopped issuing sweeps)";
        return TSP2OPT_ECUDA;
    }
    if (h->h_slot->done & 4) {
        h->has_tour = false;
        g_last_error = "device tour is not a permutation";
        return TSP2OPT_ENOTPERM;
    }
    return TSP2OPT_OK;
}

int load_device_tour(tsp2opt_ctx* h, const int32_t* d_src)
{
    h->parity = 0;
    if (++h->epoch == 0) {  // stamp wrap-around: clear and restart epochs
        CUDA_TRY(cudaMemsetAsync(h->d_stamp, 0, sizeof(unsigned) * h->n, h->stream));
        h->epoch = 1;
    }
    CUDA_TRY(launch_load_tour(h->d_coords, d_src, h->d_tour, h->d_P, h->d_E, h->n, h->d_slots + 0, h->d_stamp,
                              h->epoch, h->stream));
    if (h->nbr_k > 0) CUDA_TRY(launch_pos(h->d_tour, h->d_pos, h->n, h->stream));
    if (h->or25) CUDA_TRY(launch_gain(h->d_P, h->d_G, h->n, 0, h->n - 1, h->stream));
    h->has_tour = true;
    return TSP2OPT_OK;
}

int load_host_tour(tsp2opt_ctx* h, const int32_t* tour)
{
    int rc = validate_tour(tour, h->n);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(h->d_tour_in, tour, sizeof(int32_t) * h->n, cudaMemcpyHostToDevice, h->stream));
    return load_device_tour(h, h->d_tour_in);
}

int sweep_flags(const tsp2opt_ctx* h)
{
    return (h->seed_next && !h->first ? kSweepSeed : 0) | (h->tile_bounds != 0 ? kSweepTileBounds : 0) |
           (h->tile_bounds == 3 ? kSweepIncremental : 0) | (h->first ? kSweepFirst : 0);
}

// One iteration: sweep (a4/a5) -> allreduce-min (a6) -> apply (a7/a8).
int enqueue_iteration(tsp2opt_ctx* h, long long max_moves, bool apply)
{
    if (h->p2p && !h->p2p_ready) {
        g_last_error = "peer-memory handle used before tsp2opt_p2p_connect";
        return TSP2OPT_ESTATE;
    }
    Slot* in = h->d_slots + h->parity;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    if (h->profiling) {
        while (h->ev_pool.size() < h->ev_used + 2) {
            cudaEvent_t e;
            CUDA_TRY(cudaEventCreate(&e));
            h->ev_pool.push_back(e);
        }
        ev0 = h->ev_pool[h->ev_used];
        ev1 = h->ev_pool[h->ev_used + 1];
        h->ev_used += 2;
        CUDA_TRY(cudaEventRecord(ev0, h->stream));
    }
    const int tiling = h->or25 ? 3 : h->nbr_k > 0 ? 2 : h->tile_bounds >= 2 ? 1 : 0;
    if (h->seed_next && h->last_tiling != tiling && tiling < 2) {
        // per-tile seeds are kept per tiling: the other tiling's minima are stale
        if (tiling) CUDA_TRY(cudaMemsetAsync(h->d_ctilebest, 0xFF, sizeof(unsigned long long) * h->nctiles, h->stream));
        else CUDA_TRY(cudaMemsetAsync(h->d_tilebest, 0xFF, sizeof(unsigned long long) * h->ntiles, h->stream));
    }
    int flags = sweep_flags(h);
    // A lone sweep (best_move: no apply follows) takes the global bound -- faster on
    // incoherent tours; its minima are not reusable, so the next incremental sweep is full.
    if (!apply) flags &= ~kSweepIncremental;
    if (flags & kSweepIncremental) {  // the culled tilings (2-opt and 2.5-opt) keep per-tile minima
        const bool culled = tiling == 1 || tiling == 3;
        if (!culled || !h->inc_valid || h->last_tiling != tiling) flags |= kSweepFull;
        h->inc_valid = culled;
    } else {
        h->inc_valid = false;
    }
    h->last_tiling = tiling;
    if (tiling == 3 && h->tile_bounds >= 2 && h->cgeo.rows == kRowsSmall) {  // 2.5-opt, culled (R = 7 tiling only)
        CUDA_TRY(launch_box_cull(h->cgeo, h->d_P, h->d_E, h->d_G, h->n, h->d_ctiles, h->nctiles, h->d_rbox, h->d_cbox,
                                 h->d_list, in, apply ? 1 : 0, h->d_ctilebest, flags, h->stream));
        CUDA_TRY(launch_sweep25_list(h->cgeo, h->d_P, h->d_E, h->d_G, h->n, h->d_list, h->list25_grid, in,
                                     apply ? 1 : 0, h->d_ctilebest, flags, h->stream));
    } else if (tiling == 3) {  // 2.5-opt: dense tiling (R = 7), per-tile bound unless TILE_BOUNDS = 0
        CUDA_TRY(launch_sweep25(h->geo, h->d_P, h->d_E, h->d_G, h->n, h->d_tiles, h->ntiles, in, apply ? 1 : 0,
                                h->tile_bounds != 0 ? kSweepTileBounds : 0, h->stream));
    } else if (tiling == 2) {  // pruned neighbourhood M_K: this shard's positions, O(nK)
        const int p0 = (int)((long long)h->n * h->shard_rank / h->shard_world);
        const int p1 = (int)((long long)h->n * (h->shard_rank + 1) / h->shard_world);
        CUDA_TRY(launch_pruned_sweep(h->d_P, h->d_E, h->d_tour, h->d_pos, h->d_knn, h->nbr_k, h->n, p0, p1, in,
                                     apply ? 1 : 0, h->first, h->stream));
    } else if (tiling && (flags & kSweepIncremental) && !(flags & kSweepFull) && h->inc_fused &&
               h->cgeo.rows == kRowsSmall && h->cgeo.warps == 1 && h->inc_grid > 0) {
        // incremental: dirty tiles only, enumerated from the last move; box, cull and sweep in one launch
        CUDA_TRY(launch_inc_sweep(h->cgeo, h->d_P, h->d_E, h->n, h->d_ctiles, h->nctiles, h->d_tmap, h->inc_grid,
                                  h->d_rbox, h->d_cbox, in, apply ? 1 : 0, h->d_ctilebest, flags, h->stream));
    } else if (tiling) {  // cull first, then sweep the kept tiles only
        CUDA_TRY(launch_cull_sweep(h->cgeo, h->d_P, h->d_E, h->n, h->d_ctiles, h->nctiles, h->list_grid, h->d_rbox,
                                   h->d_cbox, h->d_list, in, apply ? 1 : 0, h->d_ctilebest, flags, h->stream));
    } else {
        CUDA_TRY(launch_sweep(h->geo, h->d_P, h->d_E, h->n, h->d_tiles, h->ntiles, in, apply ? 1 : 0, h->d_tilebest,
                              sweep_flags(h), h->stream));
    }
    if (ev1) CUDA_TRY(cudaEventRecord(ev1, h->stream));
    if (h->comm) {
        ncclResult_t r = ncclAllReduce(&in->key, &in->key, 1, ncclUint64, ncclMin, h->comm, h->stream);
        if (r != ncclSuccess) return nccl_fail(r, "ncclAllReduce");
    } else if (h->p2p) {
        CUDA_TRY(launch_p2p_min(in, h->d_peers, h->rank, h->world, apply ? 1 : 0, h->stream));
    }
    // first improvement: the min carries the marker delta; the exact delta of the winner
    if (h->first) CUDA_TRY(launch_first_fix(h->d_P, h->d_E, in, apply ? 1 : 0, h->stream));
    if (apply && h->or25) {
        Slot* out = h->d_slots + (h->parity ^ 1);
        CUDA_TRY(launch_apply25(h->d_P, h->d_E, h->d_G, h->d_tour, h->n, in, out, max_moves, 0, 0, 0, 0, h->d_trace,
                                h->d_ttype, h->trace_cap, h->d_bar25, h->stream));
        h->parity ^= 1;
    } else if (apply) {
        Slot* out = h->d_slots + (h->parity ^ 1);
        CUDA_TRY(launch_apply(h->d_P, h->d_E, h->d_tour, h->n, in, out, max_moves, 0, 0, 0, h->d_trace,
                              h->trace_cap, h->nbr_k > 0 ? h->d_pos : nullptr, h->stream));
        // dense best-improvement sweep: start the next one from the best surviving tile minimum
        if (tiling == 0 && !h->first && h->global_seed)
            CUDA_TRY(launch_global_seed(h->d_tilebest, h->ntiles, out, h->global_seed == 2 ? h->d_P : nullptr,
                                        h->global_seed == 2 ? h->d_E : nullptr, h->stream));
        h->parity ^= 1;
    }
    return TSP2OPT_OK;
}

// CUDA graphs for the multi-kernel loop (TSP2OPT_GRAPH=0 disables them).
constexpr long long kGraphBatch = 64;
constexpr double kAutoIncRho = 2.0;  // coherent tour: length < 2 sqrt(n * A) (r02_exp_c3_switch.jsonl)
bool graphs_enabled()
{
    const char* e = getenv("TSP2OPT_GRAPH");
    return !(e && atoi(e) == 0);
}

// Device-resident best-improvement loop on the loaded tour (a4-a8) until the
// local minimum or max_iters moves; leaves the final state in h->h_slot.
// Returns TSP2OPT_OK / TSP2OPT_MAXITER or a negative error.
// Workspace of the two-barrier persistent search (inc_ls2_kernel): alternate P / E / tour, its
// own tile map (which (row block, chunk) tiles of igeo exist; one GPU) and boxes, the barrier
// counter and the dense / group minima.  Allocated at creation for sizes that use it, so that no
// timed search pays for it.
static int alloc_inc2(tsp2opt_ctx* h)
{
    const size_t np = (size_t)h->n + 1 + kPad;
    const size_t wsb = inc_ls2_ws_bytes(h->igeo, h->n);
    const int TI = h->igeo.ti(), TJ = h->igeo.tj;
    const int nrb = (h->n - 1 + TI - 1) / TI, ncc = (h->n + TJ - 1) / TJ;
    std::vector<int> map((size_t)nrb * ncc, -1);
    {
        const int n = h->n;
        for (int I0 = 0, rb = 0; I0 <= n - 2; I0 += TI, rb++) {  // the tiles build_tiles keeps (pairs > 0)
            const int rows = std::min(I0 + TI, n - 1) - I0;
            for (int J0 = ((I0 + 1) / TJ) * TJ; J0 < n; J0 += TJ) {
                const int J1 = std::min(J0 + TJ, n);
                if (J1 - 1 > I0 && rows > 0) map[(size_t)rb * ncc + J0 / TJ] = 1;
            }
        }
    }
    CUDA_TRY(cudaMalloc(&h->d_P_alt, sizeof(float2) * np));
    CUDA_TRY(cudaMalloc(&h->d_E_alt, sizeof(int) * np));
    CUDA_TRY(cudaMalloc(&h->d_tour_alt, sizeof(int) * np));
    CUDA_TRY(cudaMalloc(&h->d_inc2_ws, wsb));
    CUDA_TRY(cudaMalloc(&h->d_itmap, sizeof(int) * map.size()));
    CUDA_TRY(cudaMalloc(&h->d_irbox, sizeof(Box) * (size_t)nrb));
    CUDA_TRY(cudaMalloc(&h->d_icbox, sizeof(Box) * (size_t)ncc));
    CUDA_TRY(cudaMemcpy(h->d_itmap, map.data(), sizeof(int) * map.size(), cudaMemcpyHostToDevice));
    CUDA_TRY(cudaMemset(h->d_inc2_ws, 0xFF, wsb));  // minima: none
    CUDA_TRY(cudaMalloc(&h->d_inc1_ws, inc_ls1_ws_bytes(h->igeo, h->n)));
    CUDA_TRY(cudaMemset(h->d_inc1_ws, 0xFF, inc_ls1_ws_bytes(h->igeo, h->n)));  // tile minima of tiles that
                                                                                    // do not exist: none
    return TSP2OPT_OK;
}

// Multi-kernel loop (per-iteration kernels, and sharded handles) until the local
// minimum, the move cap or, if `leave` is given, the first batch boundary where
// it returns true.  Leaves the final state in h->h_slot.
template <typename Leave>
static int run_multi_kernel_loop(tsp2opt_ctx* h, long long max_iters, const Leave* leave)
{
    int rc = 0;
    // Multi-kernel loop (and sharded handles): batches of K iterations
    // between host checks; an iteration after convergence is a no-op
    // (sweep CTAs exit on the done flag).
    // Full batches of kGraphBatch iterations are replayed from a CUDA graph
    // captured once per search (one host call instead of ~4 launches per
    // iteration); the graph starts and ends on the same slot parity.
    long long k = 4;
    cudaGraphExec_t gexec = nullptr;
    int gparity = -1;
    // Measured (profiles/r01_graph.jsonl): 2-6 % faster for the culled, pruned,
    // first-improvement and 2.5-opt loops; 20 % slower for the dense best-improvement
    // sweep (C3 from random), which keeps plain stream launches.
    const bool dense_best = !h->or25 && h->nbr_k == 0 && !h->first && h->tile_bounds < 2;
    // Sharded handles capture the ncclAllReduce into the same graph (NCCL supports
    // stream capture of collectives): one graph launch per 64 iterations on every rank.
    const bool use_graph = graphs_enabled() && !h->profiling && !dense_best;
    auto drop_graph = [&]() {
        if (gexec) cudaGraphExecDestroy(gexec);
        gexec = nullptr;
    };
    for (;;) {
        if (use_graph && k == kGraphBatch) {
            if (!gexec || gparity != h->parity) {
                drop_graph();
                gparity = h->parity;
                cudaGraph_t graph = nullptr;
                CUDA_TRY(cudaStreamBeginCapture(h->stream, cudaStreamCaptureModeThreadLocal));
                for (long long c = 0; c < k && rc == 0; c++) rc = enqueue_iteration(h, max_iters, true);
                const cudaError_t ec = cudaStreamEndCapture(h->stream, &graph);
                if (rc) {
                    if (graph) cudaGraphDestroy(graph);
                    return rc;
                }
                if (ec != cudaSuccess) return cuda_fail(ec, "cudaStreamEndCapture");
                const cudaError_t ei = cudaGraphInstantiate(&gexec, graph, 0);
                cudaGraphDestroy(graph);
                if (ei != cudaSuccess) return cuda_fail(ei, "cudaGraphInstantiate");
            }
            const cudaError_t el = cudaGraphLaunch(gexec, h->stream);
            if (el != cudaSuccess) {
                drop_graph();
                return cuda_fail(el, "cudaGraphLaunch");
            }
        } else {
            for (long long c = 0; c < k; c++) {
                rc = enqueue_iteration(h, max_iters, true);
                if (rc) return rc;
            }
        }
        rc = read_slot(h);
        if (rc) {
            drop_graph();
            return rc;
        }
        if (h->h_slot->done & 3) break;
        if (leave && (*leave)()) break;  // the caller continues with another loop
        if (k < kGraphBatch) k *= 2;
    }
    drop_graph();
    return 0;
}

int run_local_search(tsp2opt_ctx* h, long long max_iters)
{
    int rc;
    // Persistent single launch pays off while the per-iteration launch/sync
    // overhead dominates the sweep (measured: faster up to n ~ 1e3, slower from
    // n ~ 7e3 where the per-sweep kernels pack tiles better); TSP2OPT_PERSISTENT
    // = 0 / 1 forces either loop, 2 (default) chooses by pair count.
    const bool use_persistent =
        !h->comm && !h->p2p && h->nbr_k == 0 && !h->or25 && !h->first && (h->persistent == 1 || (h->persistent == 2 && h->shard_pairs <= 4000000LL));
    // dense best-improvement sweeps above that (n ~ 7e3, in-sweep tile bound): the
    // persistent loop with dynamic warp-level claims (TSP2OPT_PERSISTENT = 3 forces it)
    const bool use_dense_ls = !use_persistent && !h->comm && !h->p2p && h->nbr_k == 0 && !h->or25 && !h->first &&
                              h->tile_bounds <= 1 && h->geo.warps == 1 && !h->profiling && h->shard_world == 1 &&
                              (h->persistent == 3 || (h->persistent == 2 && h->dense_ls));
    // The incremental culled search of a single GPU in one cooperative launch per
    // ~1M iterations (launch_inc_ls2): no per-iteration launches, two grid barriers
    // per move.  Sharded handles keep the per-iteration kernels (the exchange sits
    // between sweep and apply).
    const bool inc_ok = h->inc_persistent && !h->comm && !h->p2p && h->nbr_k == 0 && !h->or25 &&
                        h->cgeo.rows == kRowsSmall && h->cgeo.warps == 1 && !h->profiling && h->shard_world == 1;
    bool use_inc_ls = inc_ok && h->tile_bounds == 3;
    // Dense loop (TILE_BOUNDS 1 by default, n ~ 7e3) until the tour is coherent, then the
    // incremental search (measured, C3: profiles/r02_exp_c3_switch.jsonl).
    const bool auto_inc = inc_ok && h->auto_inc && h->tile_bounds == 1 && !use_persistent && !use_dense_ls;
    static const double auto_rho = [] {
        const char* e = getenv("TSP2OPT_AUTO_INC_RHO");  // experiment: the hand-over threshold
        return e ? atof(e) : kAutoIncRho;
    }();
    auto coherent = [&]() { return (double)h->h_slot->length < auto_rho * h->rho_unit; };
    if (auto_inc) {
        rc = read_slot(h);
        if (rc) return rc;
        if (coherent()) use_inc_ls = true;
    }
    if (!use_inc_ls && !use_dense_ls && !use_persistent) {
        rc = run_multi_kernel_loop(h, max_iters, auto_inc ? &coherent : nullptr);
        if (rc) return rc;
        if (auto_inc && !(h->h_slot->done & 3)) use_inc_ls = true;  // left the loop: the tour became coherent
    }
    if (use_inc_ls && !(auto_inc && (h->h_slot->done & 3))) {
        const int flags = sweep_flags(h);
        // the two-barrier kernel keeps its minima in its own dense layout: tiling id 4
        const int inc_tiling = h->inc_barriers == 1 ? 5 : h->inc_barriers == 2 ? 4 : 1;
        int full = (h->inc_valid && h->last_tiling == inc_tiling) ? 0 : 1;
        for (long long launches = 0;; launches++) {
            if (launches > 1000000) {
                g_last_error = "local search did not converge";
                return TSP2OPT_ECUDA;
            }
            if (h->inc_barriers == 1) {
                const size_t np = (size_t)h->n + 1 + kPad;
                if (!h->d_P_alt) {
                    rc = alloc_inc2(h);
                    if (rc) return rc;
                }
                CUDA_TRY(launch_inc_ls1(h->igeo, h->d_P, h->d_E, h->d_tour, h->d_P_alt, h->d_E_alt, h->d_tour_alt,
                                        h->n, (int)np, h->d_itmap, h->d_inc1_ws, h->d_slots, h->parity, max_iters,
                                        1LL << 20, h->d_ctl, flags, h->d_trace, h->trace_cap, h->inc_part,
                                        h->stream));
            } else if (h->inc_barriers == 2) {
                const size_t np = (size_t)h->n + 1 + kPad;
                if (!h->d_P_alt) {
                    rc = alloc_inc2(h);
                    if (rc) return rc;
                }
                CUDA_TRY(launch_inc_ls2(h->igeo, h->d_P, h->d_E, h->d_tour, h->d_P_alt, h->d_E_alt, h->d_tour_alt,
                                        h->n, (int)np, h->d_itmap, h->d_irbox, h->d_icbox, h->d_inc2_ws, h->d_slots,
                                        h->parity, max_iters, 1LL << 20, full, h->d_ctl, flags, h->d_trace,
                                        h->trace_cap, h->inc_part, h->inc_part_bound, h->stream));
            } else {
                CUDA_TRY(launch_inc_ls(h->cgeo, h->d_P, h->d_E, h->d_tour, h->n, h->d_ctiles, h->nctiles, h->d_tmap,
                                       h->d_rbox, h->d_cbox, h->d_slots, h->parity, max_iters, 1LL << 20, full,
                                       h->d_bar, h->d_ctl, h->d_ctilebest, flags, h->d_trace, h->trace_cap,
                                       h->inc_part < 0 ? 4 : h->inc_part, h->stream));
            }
            full = 0;
            CUDA_TRY(cudaMemcpyAsync(h->h_ctl, h->d_ctl, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
            CUDA_TRY(cudaStreamSynchronize(h->stream));
            h->parity = *h->h_ctl;
            h->inc_valid = true;  // the stored tile minima are tile-local and exact for the current tour
            h->last_tiling = inc_tiling;
            rc = read_slot(h);
            if (rc) return rc;
            if (h->h_slot->done & 3) break;
        }
    } else if (use_dense_ls) {
        h->inc_valid = false;
        for (long long launches = 0;; launches++) {
            if (launches > 1000000) {
                g_last_error = "local search did not converge";
                return TSP2OPT_ECUDA;
            }
            CUDA_TRY(launch_dense_ls(h->geo, h->d_P, h->d_E, h->d_tour, h->n, h->d_tiles, h->ntiles, h->d_slots,
                                     h->parity, max_iters, 1LL << 20, h->d_bar, h->d_ctl, sweep_flags(h),
                                     h->d_tilebest, h->d_trace, h->trace_cap, h->stream));
            CUDA_TRY(cudaMemcpyAsync(h->h_ctl, h->d_ctl, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
            CUDA_TRY(cudaStreamSynchronize(h->stream));
            h->parity = *h->h_ctl;
            rc = read_slot(h);
            if (rc) return rc;
            if (h->h_slot->done & 3) break;
        }
    } else if (use_persistent) {
        h->inc_valid = false;
        // One persistent cooperative launch runs sweep -> apply to the local
        // minimum; the per-launch iteration budget bounds a launch to roughly
        // 2e12 pair checks (~0.5 s), after which the host relaunches.
        const long long pairs = std::max(1LL, h->shard_pairs);
        const long long budget = std::min(1LL << 20, std::max(16LL, 2000000000000LL / pairs));
        for (long long launches = 0;; launches++) {
            if (launches * budget > 1000LL * h->n + (1LL << 24)) {  // cannot happen: delta < 0 shortens the tour
                g_last_error = "local search did not converge";
                return TSP2OPT_ECUDA;
            }
            CUDA_TRY(launch_local_search(h->geo, h->d_P, h->d_E, h->d_tour, h->n, h->d_tiles, h->ntiles, h->d_slots,
                                         h->parity, max_iters, budget, h->d_bar, h->d_ctl, h->d_tilebest,
                                         sweep_flags(h), h->d_trace, h->trace_cap, h->stream));
            CUDA_TRY(cudaMemcpyAsync(h->h_ctl, h->d_ctl, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
            CUDA_TRY(cudaStreamSynchronize(h->stream));
            h->parity = *h->h_ctl;
            rc = read_slot(h);
            if (rc) return rc;
            if (h->h_slot->done & 3) break;
        }
    }
    return (h->h_slot->done & 3) == 2 ? TSP2OPT_MAXITER : TSP2OPT_OK;
}

int create_common(const int32_t* xy, int32_t n, int rank, int world, const void* nccl_id, bool p2p, tsp2opt_t* out)
{
    if (!out) return TSP2OPT_EINVAL;
    *out = nullptr;
    int rc = validate_coords(xy, n);
    if (rc) return rc;
    if (world < 1 || rank < 0 || rank >= world || (world > 1 && !nccl_id && !p2p)) return TSP2OPT_EINVAL;
    if (p2p && (nccl_id || world > kP2PMaxWorld)) return TSP2OPT_EINVAL;
    tsp2opt_ctx* h = new tsp2opt_ctx();
    h->n = n;
    h->rank = rank;
    h->world = world;
    auto fail = [&](int code) {
        free_ctx(h);
        return code;
    };
#define CTRY(call)                                               \
    do {                                                         \
        cudaError_t e_ = (call);                                 \
        if (e_ != cudaSuccess) return fail(cuda_fail(e_, #call)); \
    } while (0)
    CTRY(cudaGetDevice(&h->device));
    CTRY(cudaStreamCreateWithFlags(&h->own_stream, cudaStreamNonBlocking));
    h->stream = h->own_stream;
    const size_t np = (size_t)n + 1 + kPad;
    CTRY(cudaMalloc(&h->d_coords, sizeof(int) * 2 * (size_t)n));
    CTRY(cudaMalloc(&h->d_tour, sizeof(int) * np));
    CTRY(cudaMalloc(&h->d_tour_in, sizeof(int) * (size_t)n));
    CTRY(cudaMalloc(&h->d_P, sizeof(float2) * np));
    CTRY(cudaMalloc(&h->d_E, sizeof(int) * np));
    CTRY(cudaMalloc(&h->d_slots, sizeof(Slot) * 2));
    CTRY(cudaMalloc(&h->d_stamp, sizeof(unsigned) * (size_t)n));
    CTRY(cudaHostAlloc(&h->h_slot, sizeof(Slot), cudaHostAllocDefault));
    CTRY(cudaMemset(h->d_tour, 0, sizeof(int) * np));
    CTRY(cudaMemset(h->d_E, 0, sizeof(int) * np));
    CTRY(cudaMemset(h->d_stamp, 0, sizeof(unsigned) * (size_t)n));
    CTRY(cudaMalloc(&h->d_bar, sizeof(unsigned) * 2));
    CTRY(cudaMemset(h->d_bar, 0, sizeof(unsigned) * 2));
    CTRY(cudaMalloc(&h->d_ctl, sizeof(int)));
    CTRY(cudaHostAlloc(&h->h_ctl, sizeof(int), cudaHostAllocDefault));
    if (const char* ep = getenv("TSP2OPT_PERSISTENT")) h->persistent = atoi(ep);
    if (const char* es = getenv("TSP2OPT_SEED")) h->seed_next = atoi(es) != 0;
    if (const char* eg = getenv("TSP2OPT_GLOBAL_SEED")) h->global_seed = std::min(2, std::max(0, atoi(eg)));
    if (const char* ef = getenv("TSP2OPT_INC_FUSED")) h->inc_fused = atoi(ef) != 0;
    if (const char* ei = getenv("TSP2OPT_INC_PERSISTENT")) h->inc_persistent = atoi(ei) != 0;
    if (const char* eb = getenv("TSP2OPT_INC_BARRIERS")) h->inc_barriers = std::min(3, std::max(1, atoi(eb)));
    if (const char* ep2 = getenv("TSP2OPT_INC_PART")) h->inc_part = atoi(ep2);
    if (const char* eq = getenv("TSP2OPT_INC_PART_BOUND")) h->inc_part_bound = atoi(eq) != 0;
    if (const char* ed = getenv("TSP2OPT_DENSE_LS")) h->dense_ls = atoi(ed) != 0;

    CTRY(cudaMemset(h->d_slots, 0, sizeof(Slot) * 2));
    {
        std::vector<float2> pad(np, make_float2(kCoordBias, kCoordBias));
        CTRY(cudaMemcpy(h->d_P, pad.data(), sizeof(float2) * np, cudaMemcpyHostToDevice));
    }
    CTRY(cudaMemcpy(h->d_coords, xy, sizeof(int) * 2 * (size_t)n, cudaMemcpyHostToDevice));
    CTRY(sweep_prepare());
    CTRY(sweep25_prepare());
    const long long total_pairs = (long long)n * (n - 1) / 2;
    h->geo = choose_geometry(total_pairs / world);
    // Pre-sweep cull, incremental, from ~1e8 pairs per rank (measured, local search from MF:
    // n = 85900 39 vs 65 (cull) vs 212 (in-sweep bound) us per iteration, n = 33810 26 vs 36 vs
    // 79 us; n = 7397 23 vs 25 vs 18 us, where the extra launches cost more than the skipped
    // tiles; profiles/r01_ls_incremental.jsonl).
    // The level follows the instance, not the shard: a coherent tour keeps a few percent of
    // the tiles on EVERY rank, and a rank's shard of a large instance is still a spread-out
    // subset of its tiles, so C4 at 8 ranks keeps the incremental culled sweep.
    h->tile_bounds = total_pairs >= 100000000LL ? 3 : 1;
    // from ~4e6 pairs (where the per-iteration loop takes over from the persistent dense kernel)
    h->auto_inc = h->tile_bounds == 1 && total_pairs > 4000000LL;
    if (const char* eb = getenv("TSP2OPT_TILE_BOUNDS")) {
        h->tile_bounds = std::min(3, std::max(0, atoi(eb)));
        h->auto_inc = false;
    }
    if (const char* ea = getenv("TSP2OPT_AUTO_INC")) h->auto_inc = h->auto_inc && atoi(ea) != 0;
    {
        int xlo = xy[0], xhi = xy[0], ylo = xy[1], yhi = xy[1];
        for (int k = 1; k < n; k++) {
            xlo = std::min(xlo, xy[2 * k]);
            xhi = std::max(xhi, xy[2 * k]);
            ylo = std::min(ylo, xy[2 * k + 1]);
            yhi = std::max(yhi, xy[2 * k + 1]);
        }
        h->rho_unit = std::sqrt((double)n * std::max(1.0, (double)(xhi - xlo) * (double)(yhi - ylo)));
    }
    h->all_tiles = build_tiles(n, h->geo);
    // Culled-sweep tiling: R = 7 rows per lane and narrow column chunks (measured,
    // local search from MF).
    // (incremental culled sweep, measured without per-sweep events: n = 85900 TJ 32 28.6 vs 64 30.6 us
    // per iteration, n = 33810 TJ 16 20.6 vs 32 22.7 us; profiles/r01_inc_tiling.jsonl)
    // Round 2, with the persistent incremental search (one warp per kept tile, the move's cost
    // set by the slowest tile's walk): narrower chunks again -- C5 16 columns 21.9 vs 32 23.8 us
    // per move, C4 8 columns 17.7 vs 16 18.9 (profiles/r02_exp_cull_tj.jsonl).
    h->cgeo = Geometry{kRowsSmall, 1, total_pairs >= 1000000000LL ? 16 : 8};
    // The two-barrier persistent search has its own culled tiling: with kept tiles split into
    // 4-column parts over a CTA's warps and group minima, wider chunks pay again -- 32 columns from
    // 1e8 pairs: C5 Hilbert 14.6 vs 15.0 (16) / 15.5 (64) us per move, C5 MF 18.5 vs 19.8, C4 MF 15.2
    // vs 16.9 (8); C3 keeps 8 (profiles/r02_exp_inc_parts.jsonl, r02_exp_c3_inc.jsonl).  The 2.5-opt
    // and per-iteration culled sweeps keep cgeo (32 columns cost 2.5-opt at C4 35 %).
    h->igeo = Geometry{kRowsSmall, 1, total_pairs >= 100000000LL ? 32 : 8};
    if (const char* er = getenv("TSP2OPT_CULL_ROWS")) h->cgeo.rows = atoi(er) == kRowsSmall ? kRowsSmall : kRowsLarge;
    if (const char* ec = getenv("TSP2OPT_CULL_TJ"))
        if (atoi(ec) >= 2 && atoi(ec) <= kMaxTJ) h->cgeo.tj = h->igeo.tj = atoi(ec);
    if (const char* ei2 = getenv("TSP2OPT_INC_TJ"))
        if (atoi(ei2) >= 2 && atoi(ei2) <= kMaxTJ) h->igeo.tj = atoi(ei2);
    h->all_ctiles = build_tiles(n, h->cgeo);
    {
        const int nrb = (n - 1 + h->cgeo.ti() - 1) / h->cgeo.ti(), ncc = (n + h->cgeo.tj - 1) / h->cgeo.tj;
        CTRY(cudaMalloc(&h->d_rbox, sizeof(Box) * (size_t)nrb));
        CTRY(cudaMalloc(&h->d_cbox, sizeof(Box) * (size_t)ncc));
    }
    rc = upload_shard(h, rank, world);
    if (rc) return fail(rc);
    if (world == 1 && !nccl_id && !p2p && total_pairs > 4000000LL) {  // sizes that run the persistent search
        rc = alloc_inc2(h);
        if (rc) return fail(rc);
    }
    if (p2p) {  // peer-memory exchange: the mailbox now, the peers at tsp2opt_p2p_connect
        h->p2p = true;
        CTRY(cudaMalloc(&h->d_mbox, sizeof(Mailbox)));
        CTRY(cudaMemset(h->d_mbox, 0, sizeof(Mailbox)));
        CTRY(cudaMalloc(&h->d_peers, sizeof(Mailbox*) * kP2PMaxWorld));
        CTRY(cudaDeviceSynchronize());
    } else if (world > 1 || nccl_id) {  // world 1 with an id: a one-rank communicator (the sharded path on one GPU)
        ncclUniqueId id;
        memcpy(&id, nccl_id, sizeof(id));
        ncclResult_t r = ncclCommInitRank(&h->comm, world, id, rank);
        if (r != ncclSuccess) {
            h->comm = nullptr;
            return fail(nccl_fail(r, "ncclCommInitRank"));
        }
    }
#undef CTRY
    *out = h;
    return TSP2OPT_OK;
}

}  // namespace

extern "C" {

int tsp2opt_create(const int32_t* coords_xy, int32_t n, tsp2opt_t* out)
{
    return create_common(coords_xy, n, 0, 1, nullptr, false, out);
}

int tsp2opt_create_sharded(const int32_t* coords_xy, int32_t n, int32_t rank, int32_t world, const void* nccl_id,
                           tsp2opt_t* out)
{
    return create_common(coords_xy, n, rank, world, nccl_id, false, out);
}

int tsp2opt_nccl_unique_id(void* out)
{
    if (!out) return TSP2OPT_EINVAL;
    static_assert(sizeof(ncclUniqueId) == TSP2OPT_NCCL_ID_BYTES, "NCCL id size");
    ncclUniqueId id;
    ncclResult_t r = ncclGetUniqueId(&id);
    if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
    memcpy(out, &id, sizeof(id));
    return TSP2OPT_OK;
}

int tsp2opt_create_sharded_p2p(const int32_t* coords_xy, int32_t n, int32_t rank, int32_t world, tsp2opt_t* out)
{
    return create_common(coords_xy, n, rank, world, nullptr, true, out);
}

int tsp2opt_p2p_export(tsp2opt_t h, void* out)
{
    if (!h || !out || !h->p2p) return TSP2OPT_EINVAL;
    cudaIpcMemHandle_t m;
    CUDA_TRY(cudaIpcGetMemHandle(&m, h->d_mbox));
    memcpy(out, &m, sizeof(m));
    return TSP2OPT_OK;
}

int tsp2opt_p2p_connect(tsp2opt_t h, const void* handles)
{
    if (!h || !handles || !h->p2p) return TSP2OPT_EINVAL;
    if (h->p2p_ready) return TSP2OPT_ESTATE;
    std::vector<Mailbox*> peers(kP2PMaxWorld, nullptr);
    for (int r = 0; r < h->world; r++) {
        if (r == h->rank) {
            peers[r] = h->d_mbox;
            continue;
        }
        cudaIpcMemHandle_t m;
        memcpy(&m, (const char*)handles + (size_t)r * sizeof(cudaIpcMemHandle_t), sizeof(m));
        void* p = nullptr;
        const cudaError_t e = cudaIpcOpenMemHandle(&p, m, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) {
            for (void* q : h->p2p_opened) cudaIpcCloseMemHandle(q);
            h->p2p_opened.clear();
            return cuda_fail(e, "cudaIpcOpenMemHandle");
        }
        h->p2p_opened.push_back(p);
        peers[r] = (Mailbox*)p;
    }
    CUDA_TRY(cudaMemcpy(h->d_peers, peers.data(), sizeof(Mailbox*) * kP2PMaxWorld, cudaMemcpyHostToDevice));
    h->p2p_ready = true;
    return TSP2OPT_OK;
}

void tsp2opt_destroy(tsp2opt_t h)
{
    if (!h) return;
    cudaStreamSynchronize(h->stream);
    free_ctx(h);
}

int tsp2opt_set_stream(tsp2opt_t h, void* cuda_stream)
{
    if (!h) return TSP2OPT_EINVAL;
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    h->stream = cuda_stream ? (cudaStream_t)cuda_stream : h->own_stream;
    return TSP2OPT_OK;
}

int tsp2opt_set_tour(tsp2opt_t h, const int32_t* tour)
{
    if (!h || !tour) return TSP2OPT_EINVAL;
    int rc = load_host_tour(h, tour);
    if (rc) return rc;
    return read_slot(h);
}

int tsp2opt_set_tour_device_async(tsp2opt_t h, const int32_t* d_tour)
{
    if (!h || !d_tour) return TSP2OPT_EINVAL;
    return load_device_tour(h, d_tour);
}

int tsp2opt_best_move(tsp2opt_t h, const int32_t* tour, int32_t* i, int32_t* j, int32_t* delta)
{
    if (!h || !i || !j || !delta) return TSP2OPT_EINVAL;
    if (tour) {
        int rc = load_host_tour(h, tour);
        if (rc) return rc;
    }
    if (!h->has_tour) return TSP2OPT_ESTATE;
    CUDA_TRY(launch_reset_key(h->d_slots + h->parity, h->stream));
    int rc = enqueue_iteration(h, 0, false);
    if (rc) return rc;
    rc = read_slot(h);
    if (rc) return rc;
    const unsigned long long k = h->h_slot->key;
    *i = key_i(k);
    *j = key_j(k);
    *delta = key_delta(k);
    return TSP2OPT_OK;
}

int tsp2opt_apply(tsp2opt_t h, int32_t i, int32_t j)
{
    if (!h) return TSP2OPT_EINVAL;
    if (!(0 <= i && i < j && j < h->n)) return TSP2OPT_EINVAL;
    if (!h->has_tour) return TSP2OPT_ESTATE;
    Slot* in = h->d_slots + h->parity;
    Slot* out = h->d_slots + (h->parity ^ 1);
    if (h->or25)
        CUDA_TRY(launch_apply25(h->d_P, h->d_E, h->d_G, h->d_tour, h->n, in, out, 0, 1, i, j, 0, nullptr, nullptr, 0,
                                h->d_bar25, h->stream));
    else
        CUDA_TRY(launch_apply(h->d_P, h->d_E, h->d_tour, h->n, in, out, 0, 1, i, j, nullptr, 0,
                              h->nbr_k > 0 ? h->d_pos : nullptr, h->stream));
    h->parity ^= 1;
    return read_slot(h);
}

int tsp2opt_iterate_async(tsp2opt_t h, int32_t count)
{
    if (!h || count < 0) return TSP2OPT_EINVAL;
    if (!h->has_tour) return TSP2OPT_ESTATE;
    for (int c = 0; c < count; c++) {
        int rc = enqueue_iteration(h, TSP2OPT_MAX_ITERS_UNBOUNDED, true);
        if (rc) return rc;
    }
    return TSP2OPT_OK;
}

int tsp2opt_sync(tsp2opt_t h, int64_t* iterations, int64_t* length, int32_t* converged, int32_t* last_i,
                 int32_t* last_j, int32_t* last_delta)
{
    if (!h) return TSP2OPT_EINVAL;
    if (!h->has_tour) return TSP2OPT_ESTATE;
    int rc = read_slot(h);
    if (rc) return rc;
    const Slot& s = *h->h_slot;
    if (iterations) *iterations = s.moves;
    if (length) *length = s.length;
    if (converged) *converged = s.done & 3;
    if (last_i) *last_i = key_i(s.last_key);
    if (last_j) *last_j = key_j(s.last_key);
    if (last_delta) *last_delta = key_delta(s.last_key);
    return TSP2OPT_OK;
}

int tsp2opt_local_search(tsp2opt_t h, int32_t* tour, int64_t max_iters, int64_t* length, int64_t* iterations)
{
    if (!h || !length || !iterations || max_iters < 0) return TSP2OPT_EINVAL;
    int rc;
    if (tour) {
        rc = load_host_tour(h, tour);
        if (rc) return rc;
    } else {
        if (!h->has_tour) return TSP2OPT_ESTATE;
        rc = load_device_tour(h, h->d_tour);  // restart bookkeeping from the current tour
        if (rc) return rc;
    }
    rc = run_local_search(h, max_iters);
    if (rc < 0) return rc;
    if (tour) CUDA_TRY(cudaMemcpyAsync(tour, h->d_tour, sizeof(int32_t) * h->n, cudaMemcpyDeviceToHost, h->stream));
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    *length = h->h_slot->length;
    *iterations = h->h_slot->moves;
    return rc;
}

int tsp2opt_batch_local_search(const int32_t* coords_xy, int32_t n, int32_t batch, int32_t* tours,
                               int64_t max_iters, int64_t* lengths, int64_t* iterations)
{
    if (!coords_xy || !tours || !lengths || !iterations || batch < 1 || max_iters < 0) return TSP2OPT_EINVAL;
    if (n < 3 || n > kBatchMaxN) return TSP2OPT_EINVAL;
    for (long long b = 0; b < batch; b++) {
        int rc = validate_coords(coords_xy + 2 * n * b, n);
        if (rc) return rc;
        rc = validate_tour(tours + (long long)n * b, n);
        if (rc) return rc;
    }
    int* d_xy = nullptr;
    int* d_t = nullptr;
    long long* d_out = nullptr;
    auto cleanup = [&]() {
        cudaFree(d_xy);
        cudaFree(d_t);
        cudaFree(d_out);
    };
    auto fail = [&](cudaError_t e, const char* what) {
        cleanup();
        return cuda_fail(e, what);
    };
    const size_t nxy = sizeof(int) * 2 * (size_t)n * batch, nt = sizeof(int) * (size_t)n * batch;
    cudaError_t e;
    if ((e = cudaMalloc(&d_xy, nxy)) != cudaSuccess) return fail(e, "cudaMalloc");
    if ((e = cudaMalloc(&d_t, nt)) != cudaSuccess) return fail(e, "cudaMalloc");
    if ((e = cudaMalloc(&d_out, sizeof(long long) * 2 * (size_t)batch)) != cudaSuccess) return fail(e, "cudaMalloc");
    if ((e = cudaMemcpy(d_xy, coords_xy, nxy, cudaMemcpyHostToDevice)) != cudaSuccess) return fail(e, "H2D");
    if ((e = cudaMemcpy(d_t, tours, nt, cudaMemcpyHostToDevice)) != cudaSuccess) return fail(e, "H2D");
    if ((e = launch_batch_local_search(d_xy, d_t, n, batch, max_iters, d_out, d_out + batch, nullptr)) != cudaSuccess)
        return fail(e, "batch_ls_kernel");
    if ((e = cudaMemcpy(tours, d_t, nt, cudaMemcpyDeviceToHost)) != cudaSuccess) return fail(e, "D2H");
    std::vector<long long> out(2 * (size_t)batch);
    if ((e = cudaMemcpy(out.data(), d_out, sizeof(long long) * out.size(), cudaMemcpyDeviceToHost)) != cudaSuccess)
        return fail(e, "D2H");
    cleanup();
    for (int b = 0; b < batch; b++)
        if (out[b] < 0) return TSP2OPT_ENOTPERM;  // unreachable: validated above
    for (int b = 0; b < batch; b++) {
        lengths[b] = out[b];
        iterations[b] = out[batch + b];
    }
    return TSP2OPT_OK;
}

int tsp2opt_batch_local_search_async(const int32_t* d_coords_xy, int32_t n, int32_t batch, int32_t* d_tours,
                                     int64_t max_iters, int64_t* d_lengths, int64_t* d_iterations, void* stream)
{
    if (!d_coords_xy || !d_tours || !d_lengths || !d_iterations || batch < 1 || max_iters < 0) return TSP2OPT_EINVAL;
    if (n < 3 || n > kBatchMaxN) return TSP2OPT_EINVAL;
    const cudaError_t e = launch_batch_local_search(d_coords_xy, d_tours, n, batch, max_iters,
                                                    reinterpret_cast<long long*>(d_lengths),
                                                    reinterpret_cast<long long*>(d_iterations),
                                                    static_cast<cudaStream_t>(stream));
    return e == cudaSuccess ? TSP2OPT_OK : cuda_fail(e, "batch_ls_kernel");
}

int tsp2opt_batch_ils(const int32_t* coords_xy, int32_t n, int32_t batch, int32_t* tours, int64_t iterations,
                      const uint64_t* seeds, int64_t* lengths, int64_t* history)
{
    if (!coords_xy || !tours || !seeds || !lengths || batch < 1 || iterations < 0) return TSP2OPT_EINVAL;
    if (n < 3 || n > kBatchMaxN) return TSP2OPT_EINVAL;
    for (long long b = 0; b < batch; b++) {
        int rc = validate_coords(coords_xy + 2 * n * b, n);
        if (rc) return rc;
        rc = validate_tour(tours + (long long)n * b, n);
        if (rc) return rc;
    }
    const size_t nxy = sizeof(int) * 2 * (size_t)n * batch, nt = sizeof(int) * (size_t)n * batch;
    const size_t nh = history ? sizeof(long long) * (size_t)(iterations + 1) * batch : 0;
    int* d_xy = nullptr;
    int* d_t = nullptr;
    unsigned long long* d_seed = nullptr;
    long long* d_len = nullptr;
    long long* d_hist = nullptr;
    auto cleanup = [&]() {
        cudaFree(d_xy);
        cudaFree(d_t);
        cudaFree(d_seed);
        cudaFree(d_len);
        cudaFree(d_hist);
    };
    auto fail = [&](cudaError_t e, const char* what) {
        cleanup();
        return cuda_fail(e, what);
    };
    cudaError_t e;
    if ((e = cudaMalloc(&d_xy, nxy)) != cudaSuccess) return fail(e, "cudaMalloc");
    if ((e = cudaMalloc(&d_t, nt)) != cudaSuccess) return fail(e, "cudaMalloc");
    if ((e = cudaMalloc(&d_seed, sizeof(uint64_t) * batch)) != cudaSuccess) return fail(e, "cudaMalloc");
    if ((e = cudaMalloc(&d_len, sizeof(long long) * batch)) != cudaSuccess) return fail(e, "cudaMalloc");
    if (nh && (e = cudaMalloc(&d_hist, nh)) != cudaSuccess) return fail(e, "cudaMalloc");
    if ((e = cudaMemcpy(d_xy, coords_xy, nxy, cudaMemcpyHostToDevice)) != cudaSuccess) return fail(e, "H2D");
    if ((e = cudaMemcpy(d_t, tours, nt, cudaMemcpyHostToDevice)) != cudaSuccess) return fail(e, "H2D");
    if ((e = cudaMemcpy(d_seed, seeds, sizeof(uint64_t) * batch, cudaMemcpyHostToDevice)) != cudaSuccess)
        return fail(e, "H2D");
    if ((e = launch_batch_ils(d_xy, d_t, n, batch, iterations, d_seed, d_len, d_hist, nullptr)) != cudaSuccess)
        return fail(e, "batch_ils_kernel");
    if ((e = cudaMemcpy(tours, d_t, nt, cudaMemcpyDeviceToHost)) != cudaSuccess) return fail(e, "D2H");
    if ((e = cudaMemcpy(lengths, d_len, sizeof(long long) * batch, cudaMemcpyDeviceToHost)) != cudaSuccess)
        return fail(e, "D2H");
    if (nh && (e = cudaMemcpy(history, d_hist, nh, cudaMemcpyDeviceToHost)) != cudaSuccess) return fail(e, "D2H");
    cleanup();
    return TSP2OPT_OK;
}

int tsp2opt_batch_ils_async(const int32_t* d_coords_xy, int32_t n, int32_t batch, int32_t* d_tours,
                            int64_t iterations, const uint64_t* d_seeds, int64_t* d_lengths, int64_t* d_history,
                            void* stream)
{
    if (!d_coords_xy || !d_tours || !d_seeds || !d_lengths || batch < 1 || iterations < 0) return TSP2OPT_EINVAL;
    if (n < 3 || n > kBatchMaxN) return TSP2OPT_EINVAL;
    const cudaError_t e = launch_batch_ils(d_coords_xy, d_tours, n, batch, iterations,
                                           reinterpret_cast<const unsigned long long*>(d_seeds),
                                           reinterpret_cast<long long*>(d_lengths),
                                           reinterpret_cast<long long*>(d_history), static_cast<cudaStream_t>(stream));
    return e == cudaSuccess ? TSP2OPT_OK : cuda_fail(e, "batch_ils_kernel");
}

int tsp2opt_ils(tsp2opt_t h, int32_t* tour, int64_t iterations, uint64_t seed, int64_t* length, int64_t* lengths)
{
    if (!h || !tour || !length || iterations < 0) return TSP2OPT_EINVAL;
    // The local search of each step is the handle's: 2-opt, pruned (R18), first
    // improvement (R20) or 2.5-opt (R19) -- oracle_ils_mode
    int rc = load_host_tour(h, tour);
    if (rc) return rc;
    if (!h->d_best) CUDA_TRY(cudaMalloc(&h->d_best, sizeof(int) * (size_t)h->n));
    // s* = 2optLocalSearch(s0)
    rc = run_local_search(h, TSP2OPT_MAX_ITERS_UNBOUNDED);
    if (rc < 0) return rc;
    long long best = h->h_slot->length;
    CUDA_TRY(cudaMemcpyAsync(h->d_best, h->d_tour, sizeof(int) * (size_t)h->n, cudaMemcpyDeviceToDevice, h->stream));
    if (lengths) lengths[0] = best;
    for (long long t = 0; t < iterations; t++) {
        if (h->n >= 8) {
            // s' = Perturbation(s*): double bridge of the best tour (device gather),
            // s*' = 2optLocalSearch(s'), accept iff strictly shorter (R14-R16)
            long long a, b, c;
            ils_cuts(h->n, seed, t, &a, &b, &c);
            CUDA_TRY(launch_double_bridge(h->d_best, h->d_tour_in, h->n, (int)a, (int)b, (int)c, h->stream));
            rc = load_device_tour(h, h->d_tour_in);
            if (rc) return rc;
            rc = run_local_search(h, TSP2OPT_MAX_ITERS_UNBOUNDED);
            if (rc < 0) return rc;
            if (h->h_slot->length < best) {
                best = h->h_slot->length;
                CUDA_TRY(cudaMemcpyAsync(h->d_best, h->d_tour, sizeof(int) * (size_t)h->n, cudaMemcpyDeviceToDevice,
                                         h->stream));
            }
        }
        if (lengths) lengths[t + 1] = best;
    }
    // leave the handle holding the best tour
    CUDA_TRY(cudaMemcpyAsync(h->d_tour_in, h->d_best, sizeof(int) * (size_t)h->n, cudaMemcpyDeviceToDevice,
                             h->stream));
    rc = load_device_tour(h, h->d_tour_in);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(tour, h->d_best, sizeof(int32_t) * h->n, cudaMemcpyDeviceToHost, h->stream));
    rc = read_slot(h);
    if (rc) return rc;
    *length = best;
    return TSP2OPT_OK;
}

int tsp2opt_mf_tour(tsp2opt_t h, int32_t* tour_out, int64_t* length, int32_t* rounds)
{
    if (!h) return TSP2OPT_EINVAL;
    if (!h->d_mf_ws) CUDA_TRY(cudaMalloc(&h->d_mf_ws, mf_workspace_bytes(h->n)));
    CUDA_TRY(launch_mf_tour(h->d_coords, h->n, h->d_mf_ws, h->d_tour_in, &h->mf_rounds, h->stream));
    int rc = load_device_tour(h, h->d_tour_in);
    if (rc) return rc;
    rc = read_slot(h);  // also proves the ranked tour is a permutation
    if (rc) return rc;
    if (tour_out) {
        CUDA_TRY(cudaMemcpyAsync(tour_out, h->d_tour, sizeof(int32_t) * h->n, cudaMemcpyDeviceToHost, h->stream));
        CUDA_TRY(cudaStreamSynchronize(h->stream));
    }
    if (length) *length = h->h_slot->length;
    if (rounds) *rounds = h->mf_rounds;
    return TSP2OPT_OK;
}

int tsp2opt_get_tour(tsp2opt_t h, int32_t* tour_out, int64_t* length)
{
    if (!h || !tour_out) return TSP2OPT_EINVAL;
    if (!h->has_tour) return TSP2OPT_ESTATE;
    int rc = read_slot(h);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(tour_out, h->d_tour, sizeof(int32_t) * h->n, cudaMemcpyDeviceToHost, h->stream));
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    if (length) *length = h->h_slot->length;
    return TSP2OPT_OK;
}

int tsp2opt_set_option(tsp2opt_t h, int32_t option, int64_t value)
{
    if (!h) return TSP2OPT_EINVAL;
    h->inc_valid = false;  // any option change: the next incremental sweep starts from scratch
    switch (option) {
    case TSP2OPT_OPT_TILE_BOUNDS:
        if (value < 0 || value > 3) return TSP2OPT_EINVAL;
        h->tile_bounds = (int)value;
        h->auto_inc = false;
        break;
    case TSP2OPT_OPT_SEED: h->seed_next = value != 0; break;
    case TSP2OPT_OPT_TRACE: {
        if (value < 0) return TSP2OPT_EINVAL;
        CUDA_TRY(cudaStreamSynchronize(h->stream));
        cudaFree(h->d_trace);
        cudaFree(h->d_ttype);
        h->d_trace = nullptr;
        h->d_ttype = nullptr;
        h->trace_cap = 0;
        if (value > 0) {
            CUDA_TRY(cudaMalloc(&h->d_trace, sizeof(unsigned long long) * (size_t)value));
            CUDA_TRY(cudaMalloc(&h->d_ttype, sizeof(int) * (size_t)value));
            CUDA_TRY(cudaMemset(h->d_ttype, 0, sizeof(int) * (size_t)value));
            h->trace_cap = value;
        }
        break;
    }
    case TSP2OPT_OPT_PERSISTENT:
        if (value < 0 || value > 2) return TSP2OPT_EINVAL;
        h->persistent = (int)value;
        break;
    case TSP2OPT_OPT_FIRST_IMPROVEMENT: {
        if (value < 0 || value > 1 || (value && h->or25)) return TSP2OPT_EINVAL;
        h->first = (int)value;
        if (h->has_tour) CUDA_TRY(launch_reset_key(h->d_slots + h->parity, h->stream));  // pending key: other rule
        CUDA_TRY(cudaStreamSynchronize(h->stream));
        break;
    }
    case TSP2OPT_OPT_NODE_INSERTION: {
        if (value < 0 || value > 1 || (value && (h->nbr_k > 0 || h->first))) return TSP2OPT_EINVAL;
        CUDA_TRY(cudaStreamSynchronize(h->stream));
        if (value && !h->d_G) {
            const size_t np = (size_t)h->n + 1 + kPad;
            CUDA_TRY(cudaMalloc(&h->d_G, sizeof(int) * np));
            CUDA_TRY(cudaMemset(h->d_G, 0, sizeof(int) * np));
            CUDA_TRY(cudaMalloc(&h->d_bar25, sizeof(unsigned) * 2));
            CUDA_TRY(cudaMemset(h->d_bar25, 0, sizeof(unsigned) * 2));
        }
        // the 2.5-opt sweep is instantiated for R = 7 only; the 2-opt geometry comes back with value 0
        const long long total_pairs = (long long)h->n * (h->n - 1) / 2;
        Geometry g = choose_geometry(total_pairs / h->world);
        if (value) g.rows = kRowsSmall;
        if (g.rows != h->geo.rows || g.tj != h->geo.tj || g.warps != h->geo.warps) {
            h->geo = g;
            h->all_tiles = build_tiles(h->n, h->geo);
            int rc = upload_shard(h, h->shard_rank, h->shard_world);
            if (rc) return rc;
        }
        h->or25 = (int)value;
        if (h->has_tour) {
            if (value) CUDA_TRY(launch_gain(h->d_P, h->d_G, h->n, 0, h->n - 1, h->stream));
            CUDA_TRY(launch_reset_key(h->d_slots + h->parity, h->stream));
        }
        h->last_tiling = -1;
        CUDA_TRY(cudaStreamSynchronize(h->stream));
        break;
    }
    case TSP2OPT_OPT_NEIGHBOURS: {
        if (value < 0 || value > kMaxNeighbours || (value && h->or25)) return TSP2OPT_EINVAL;
        if (value > 0) {
            if (!h->d_knn) {  // exact candidate lists, once per handle (coordinates never change)
                unsigned long long* knn = nullptr;
                CUDA_TRY(cudaMalloc(&knn, sizeof(unsigned long long) * kMaxNeighbours * (size_t)h->n));
                h->d_knn = knn;
                CUDA_TRY(launch_knn(h->d_coords, h->n, h->d_knn, h->stream));
            }
            if (!h->d_pos) CUDA_TRY(cudaMalloc(&h->d_pos, sizeof(int) * (size_t)h->n));
            if (h->has_tour) CUDA_TRY(launch_pos(h->d_tour, h->d_pos, h->n, h->stream));
        }
        // the pending key may be a pair of the other neighbourhood: restart it from the seed
        if (h->has_tour) CUDA_TRY(launch_reset_key(h->d_slots + h->parity, h->stream));
        CUDA_TRY(cudaStreamSynchronize(h->stream));
        h->nbr_k = (int)value;
        h->last_tiling = -1;  // per-tile seeds of a dense sweep are stale after pruned moves
        break;
    }
    default: return TSP2OPT_EINVAL;
    }
    return TSP2OPT_OK;
}

int tsp2opt_get_trace(tsp2opt_t h, int32_t* ijd, int64_t cap, int64_t* count)
{
    if (!h || !count || (cap > 0 && !ijd)) return TSP2OPT_EINVAL;
    if (!h->has_tour) return TSP2OPT_ESTATE;
    int rc = read_slot(h);
    if (rc) return rc;
    const long long k = std::min<long long>(h->h_slot->moves, h->trace_cap);
    *count = k;
    const long long m = std::min<long long>(k, cap);
    if (m > 0) {
        std::vector<unsigned long long> keys((size_t)m);
        CUDA_TRY(cudaMemcpy(keys.data(), h->d_trace, sizeof(unsigned long long) * (size_t)m, cudaMemcpyDeviceToHost));
        for (long long t = 0; t < m; t++) {
            ijd[3 * t] = key_i(keys[t]);
            ijd[3 * t + 1] = key_j(keys[t]);
            ijd[3 * t + 2] = key_delta(keys[t]);
        }
    }
    return TSP2OPT_OK;
}

int tsp2opt_get_trace_typed(tsp2opt_t h, int32_t* ijdt, int64_t cap, int64_t* count)
{
    if (!h || !count || (cap > 0 && !ijdt)) return TSP2OPT_EINVAL;
    if (!h->has_tour) return TSP2OPT_ESTATE;
    int rc = read_slot(h);
    if (rc) return rc;
    const long long k = std::min<long long>(h->h_slot->moves, h->trace_cap);
    *count = k;
    const long long m = std::min<long long>(k, cap);
    if (m > 0) {
        std::vector<unsigned long long> keys((size_t)m);
        std::vector<int> types((size_t)m);
        CUDA_TRY(cudaMemcpy(keys.data(), h->d_trace, sizeof(unsigned long long) * (size_t)m, cudaMemcpyDeviceToHost));
        CUDA_TRY(cudaMemcpy(types.data(), h->d_ttype, sizeof(int) * (size_t)m, cudaMemcpyDeviceToHost));
        for (long long t = 0; t < m; t++) {
            ijdt[4 * t] = key_i(keys[t]);
            ijdt[4 * t + 1] = key_j(keys[t]);
            ijdt[4 * t + 2] = key_delta(keys[t]);
            ijdt[4 * t + 3] = h->or25 ? types[t] : 0;
        }
    }
    return TSP2OPT_OK;
}

int tsp2opt_best_move_typed(tsp2opt_t h, const int32_t* tour, int32_t* i, int32_t* j, int32_t* type, int32_t* delta)
{
    if (!h || !i || !j || !type || !delta) return TSP2OPT_EINVAL;
    if (tour) {
        int rc = load_host_tour(h, tour);
        if (rc) return rc;
    }
    if (!h->has_tour) return TSP2OPT_ESTATE;
    CUDA_TRY(launch_reset_key(h->d_slots + h->parity, h->stream));
    int rc = enqueue_iteration(h, 0, false);
    if (rc) return rc;
    if (h->or25) CUDA_TRY(launch_decide25(h->d_P, h->d_E, h->d_G, h->d_slots + h->parity, h->stream));
    rc = read_slot(h);
    if (rc) return rc;
    const unsigned long long k = h->h_slot->key;
    *i = key_i(k);
    *j = key_j(k);
    *delta = key_delta(k);
    *type = h->or25 ? h->h_slot->mtype : 0;
    return TSP2OPT_OK;
}

int tsp2opt_apply_typed(tsp2opt_t h, int32_t i, int32_t j, int32_t type)
{
    if (!h || type < 0 || type > 2) return TSP2OPT_EINVAL;
    if (type == 0) return tsp2opt_apply(h, i, j);
    if (!h->or25 || !(0 <= i && i + 2 <= j && j < h->n)) return TSP2OPT_EINVAL;
    if (!h->has_tour) return TSP2OPT_ESTATE;
    Slot* in = h->d_slots + h->parity;
    Slot* out = h->d_slots + (h->parity ^ 1);
    CUDA_TRY(launch_apply25(h->d_P, h->d_E, h->d_G, h->d_tour, h->n, in, out, 0, 1, i, j, type, nullptr, nullptr, 0,
                            h->d_bar25, h->stream));
    h->parity ^= 1;
    return read_slot(h);
}

int tsp2opt_debug_set_shard(tsp2opt_t h, int32_t rank, int32_t world)
{
    if (!h || world < 1 || rank < 0 || rank >= world) return TSP2OPT_EINVAL;
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    return upload_shard(h, rank, world);
}

int tsp2opt_plan_shard(int32_t n, int32_t rank, int32_t world, int32_t* R, int32_t* warps, int32_t* tj,
                       int32_t* tiles_out, int64_t cap, int64_t* ntiles, int64_t* pairs)
{
    if (n < 3 || n > TSP2OPT_MAX_N || world < 1 || rank < 0 || rank >= world || !ntiles || !pairs)
        return TSP2OPT_EINVAL;
    const Geometry g = choose_geometry((long long)n * (n - 1) / 2 / world);
    long long p = 0;
    std::vector<Tile> mine = shard_tiles(build_tiles(n, g), rank, world, &p);
    if (R) *R = g.rows;
    if (warps) *warps = g.warps;
    if (tj) *tj = g.tj;
    *ntiles = (int64_t)mine.size();
    *pairs = p;
    if (tiles_out)
        for (size_t k = 0; k < mine.size() && (int64_t)k < cap; k++) {
            tiles_out[2 * k] = mine[k].i0;
            tiles_out[2 * k + 1] = mine[k].j0;
        }
    return TSP2OPT_OK;
}

int tsp2opt_get_geometry(tsp2opt_t h, int32_t* R, int32_t* warps, int32_t* tj, int64_t* tiles, int64_t* pairs)
{
    if (!h) return TSP2OPT_EINVAL;
    if (R) *R = h->geo.rows;
    if (warps) *warps = h->geo.warps;
    if (tj) *tj = h->geo.tj;
    if (tiles) *tiles = h->ntiles;
    if (pairs) *pairs = h->shard_pairs;
    return TSP2OPT_OK;
}

int tsp2opt_selftest(int64_t* dist_violations, int64_t* filter_violations, int64_t* first_bad_s,
                     int64_t* first_bad_dxdy)
{
    if (!dist_violations || !filter_violations) return TSP2OPT_EINVAL;
    long long r[4] = {-1, -1, -1, -1};
    CUDA_TRY(run_selftest(r));
    *dist_violations = r[0];
    *filter_violations = r[1];
    if (first_bad_s) *first_bad_s = r[0] ? r[2] : -1;
    if (first_bad_dxdy) *first_bad_dxdy = r[1] ? r[3] : -1;
    return TSP2OPT_OK;
}

int tsp2opt_profile(tsp2opt_t h, int32_t enable)
{
    if (!h) return TSP2OPT_EINVAL;
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    h->profiling = enable != 0;
    h->ev_used = 0;
    return TSP2OPT_OK;
}

int tsp2opt_profile_read(tsp2opt_t h, double* total_ms, int64_t* launches)
{
    if (!h || !total_ms || !launches) return TSP2OPT_EINVAL;
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    double sum = 0;
    for (size_t k = 0; k + 1 < h->ev_used; k += 2) {
        float ms = 0;
        CUDA_TRY(cudaEventElapsedTime(&ms, h->ev_pool[k], h->ev_pool[k + 1]));
        sum += ms;
    }
    *total_ms = sum;
    *launches = (int64_t)(h->ev_used / 2);
    return TSP2OPT_OK;
}

int64_t tsp2opt_launch_count(void) { return launch_count(); }

int tsp2opt_selftest_sqrt(double* max_rel_err, int32_t* zero_ok)
{
    if (!max_rel_err || !zero_ok) return TSP2OPT_EINVAL;
    int z = 0;
    CUDA_TRY(run_selftest_sqrt(max_rel_err, &z));
    *zero_ok = z;
    return TSP2OPT_OK;
}

int tsp2opt_debug_phases(int64_t* out16, int32_t reset)
{
    if (!out16) return TSP2OPT_EINVAL;
    long long v[16];
    CUDA_TRY(read_phases(v, reset));
    for (int k = 0; k < 16; k++) out16[k] = v[k];
    return TSP2OPT_OK;
}

int tsp2opt_debug_stats(int64_t* out4, int32_t reset)
{
    if (!out4) return TSP2OPT_EINVAL;
    long long r[4];
    CUDA_TRY(cudaDeviceSynchronize());
    CUDA_TRY(read_stats(r, reset));
    for (int k = 0; k < 4; k++) out4[k] = r[k];
    return TSP2OPT_OK;
}

const char* tsp2opt_strerror(int code)
{
    switch (code) {
    case TSP2OPT_OK: return "ok";
    case TSP2OPT_MAXITER: return "max_iters reached with an improving move left";
    case TSP2OPT_EINVAL: return "invalid argument";
    case TSP2OPT_ERANGE: return "coordinate outside [0, 2^15)";
    case TSP2OPT_ENOTPERM: return "tour is not a permutation of 0..n-1";
    case TSP2OPT_ESTATE: return "no tour loaded";
    case TSP2OPT_ECUDA: return "CUDA error";
    case TSP2OPT_ENCCL: return "NCCL error";
    case TSP2OPT_ENOMEM: return "out of memory";
    default: return "unknown error";
    }
}

const char* tsp2opt_last_error(void) { return g_last_error.c_str(); }

}  // extern "C"

// ---------------------------------------------------------------------------
// Or-opt (reading R21; tsp2opt_oropt.cu).  Stateless:
// upload, then per move one dense sweep, an 8-byte key read and the apply.
namespace {

int or_run(const int32_t* coords_xy, int32_t n, int32_t* tour, int64_t max_iters, int64_t* length,
           int64_t* iterations, int32_t* trace, int64_t trace_cap, unsigned long long* first_key)
{
    int rc = validate_coords(coords_xy, n);
    if (rc) return rc;
    rc = validate_tour(tour, n);
    if (rc) return rc;
    int* d_xy = nullptr;
    int* d_t = nullptr;
    int* d_span = nullptr;
    int* d_trace = nullptr;
    int2* d_q = nullptr;
    int4* d_c = nullptr;  // per-position sweep constants CR | CC
    unsigned long long* d_slot = nullptr;  // kOrSlotWords: key, length, moves, done, cap, move
    unsigned long long h_slot[kOrSlotWords] = {};  // readback (pageable: a pinned buffer costs ~1 ms per call)
    cudaStream_t st = nullptr;
    cudaGraphExec_t gexec = nullptr;
    auto cleanup = [&]() {
        if (gexec) cudaGraphExecDestroy(gexec);
        if (st) cudaStreamDestroy(st);
        cudaFree(d_c);
        cudaFree(d_xy);
        cudaFree(d_t);
        cudaFree(d_span);
        cudaFree(d_trace);
        cudaFree(d_q);
        cudaFree(d_slot);
    };
    auto fail = [&](cudaError_t e, const char* what) {
        cleanup();
        return cuda_fail(e, what);
    };
    cudaError_t e;
    const size_t nb = sizeof(int) * (size_t)n;
    const long long tcap = trace ? std::min<long long>(trace_cap, max_iters) : 0;
    if ((e = cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking)) != cudaSuccess) return fail(e, "stream");
    if ((e = cudaMalloc(&d_xy, 2 * nb)) != cudaSuccess) return fail(e, "cudaMalloc");
    if ((e = cudaMalloc(&d_t, nb)) != cudaSuccess) return fail(e, "cudaMalloc");
    if ((e = cudaMalloc(&d_span, nb)) != cudaSuccess) return fail(e, "cudaMalloc");
    if (tcap > 0 && (e = cudaMalloc(&d_trace, sizeof(int) * 4 * (size_t)tcap)) != cudaSuccess)
        return fail(e, "cudaMalloc");
    if ((e = cudaMalloc(&d_q, sizeof(int2) * oropt_q_entries(n))) != cudaSuccess) return fail(e, "cudaMalloc");
    if ((e = cudaMalloc(&d_slot, kOrSlotWords * sizeof(unsigned long long))) != cudaSuccess) return fail(e, "cudaMalloc");
    if ((e = cudaMalloc(&d_c, 2 * sizeof(int4) * oropt_const_entries(n))) != cudaSuccess) return fail(e, "cudaMalloc");
    {
        unsigned long long init[kOrSlotWords] = {};
        init[kOrCap] = (unsigned long long)max_iters;
        if ((e = cudaMemcpyAsync(d_slot, init, sizeof(init), cudaMemcpyHostToDevice, st)) != cudaSuccess)
            return fail(e, "H2D");
        if ((e = cudaMemcpyAsync(d_xy, coords_xy, 2 * nb, cudaMemcpyHostToDevice, st)) != cudaSuccess)
            return fail(e, "H2D");
        if ((e = cudaMemcpyAsync(d_t, tour, nb, cudaMemcpyHostToDevice, st)) != cudaSuccess) return fail(e, "H2D");
        if ((e = launch_or_load(d_xy, d_t, d_q, n, d_slot + kOrLength, st)) != cudaSuccess) return fail(e, "or_load");
        if ((e = cudaStreamSynchronize(st)) != cudaSuccess) return fail(e, "sync");
    }
    // Device-resident loop (no host decision per move): each iteration is the sweep
    // (constants + tile kernel), the decide kernel and the apply; batches of k
    // iterations between host reads of the state, k doubling to 64, full batches
    // replayed from one captured CUDA graph.  An iteration after convergence is a no-op.
    auto enqueue = [&](long long k) -> cudaError_t {
        for (long long c = 0; c < k; c++) {
            cudaError_t x = launch_or_sweep(d_q, d_c, d_c + oropt_const_entries(n), n, d_slot, st);
            if (x == cudaSuccess) x = launch_or_apply(d_xy, d_t, d_q, d_span, n, d_slot, d_trace, tcap, st);
            if (x != cudaSuccess) return x;
        }
        return cudaSuccess;
    };
    long long k = 1, full_batches = 0;
    for (long long batches = 0;; batches++) {
        if (batches > (1LL << 26)) return fail(cudaErrorUnknown, "Or-opt local search did not converge");
        // (below n = 512 an iteration is a few microseconds: capturing costs more than it saves)
        if (k == 64 && n >= 512 && graphs_enabled() && ++full_batches >= 1) {
            if (!gexec) {
                cudaGraph_t graph = nullptr;
                if ((e = cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal)) != cudaSuccess)
                    return fail(e, "capture");
                const cudaError_t eq = enqueue(k);
                e = cudaStreamEndCapture(st, &graph);
                if (eq != cudaSuccess) {
                    if (graph) cudaGraphDestroy(graph);
                    return fail(eq, "Or-opt iteration");
                }
                if (e != cudaSuccess) return fail(e, "capture");
                e = cudaGraphInstantiate(&gexec, graph, 0);
                cudaGraphDestroy(graph);
                if (e != cudaSuccess) return fail(e, "cudaGraphInstantiate");
            }
            if ((e = cudaGraphLaunch(gexec, st)) != cudaSuccess) return fail(e, "cudaGraphLaunch");
        } else if ((e = enqueue(k)) != cudaSuccess) {
            return fail(e, "Or-opt iteration");
        }
        if ((e = cudaMemcpyAsync(h_slot, d_slot, kOrSlotWords * sizeof(unsigned long long), cudaMemcpyDeviceToHost,
                                 st)) != cudaSuccess)
            return fail(e, "D2H");
        if ((e = cudaStreamSynchronize(st)) != cudaSuccess) return fail(e, "sync");
        if (first_key && batches == 0) *first_key = h_slot[0];  // the first sweep's key (best_move: max_iters 0)
        if (h_slot[kOrDone]) break;
        if (k < 64) k *= 2;
    }
    const int status = h_slot[kOrDone] == 2 ? TSP2OPT_MAXITER : TSP2OPT_OK;
    const long long it = (long long)h_slot[kOrMoves], L = (long long)h_slot[kOrLength];
    std::vector<int32_t> tr(4 * (size_t)std::min<long long>(it, tcap));
    if (!tr.empty() && (e = cudaMemcpy(tr.data(), d_trace, sizeof(int32_t) * tr.size(), cudaMemcpyDeviceToHost)) !=
                           cudaSuccess)
        return fail(e, "D2H");
    std::vector<int32_t> out(n);
    if ((e = cudaMemcpy(out.data(), d_t, nb, cudaMemcpyDeviceToHost)) != cudaSuccess) return fail(e, "D2H");
    cleanup();
    // nothing is written to the caller before this point (errors leave tour / trace untouched)
    memcpy(tour, out.data(), nb);
    if (!tr.empty()) memcpy(trace, tr.data(), sizeof(int32_t) * tr.size());
    if (length) *length = L;
    if (iterations) *iterations = it;
    return status;
}

}  // namespace

int tsp2opt_oropt_local_search(const int32_t* coords_xy, int32_t n, int32_t* tour, int64_t max_iters,
                               int64_t* length, int64_t* iterations, int32_t* trace_ijdt, int64_t trace_cap)
{
    if (!coords_xy || !tour || max_iters < 0 || trace_cap < 0 || (trace_cap > 0 && !trace_ijdt)) return TSP2OPT_EINVAL;
    if (n < 3 || n > TSP2OPT_OROPT_MAX_N) return TSP2OPT_EINVAL;
    return or_run(coords_xy, n, tour, max_iters, length, iterations, trace_ijdt, trace_cap, nullptr);
}

int tsp2opt_oropt_config(int32_t filter, int32_t naive)
{
    if (filter < -1 || filter > 1 || naive < 0 || naive > 1) return TSP2OPT_EINVAL;
    or_config(filter, naive);
    return TSP2OPT_OK;
}

int tsp2opt_oropt_best_move(const int32_t* coords_xy, int32_t n, const int32_t* tour, int32_t* i, int32_t* j,
                            int32_t* type, int32_t* delta)
{
    if (!coords_xy || !tour || !i || !j || !type || !delta) return TSP2OPT_EINVAL;
    if (n < 3 || n > TSP2OPT_OROPT_MAX_N) return TSP2OPT_EINVAL;
    std::vector<int32_t> t(tour, tour + n);
    unsigned long long key = 0;
    int rc = or_run(coords_xy, n, t.data(), 0, nullptr, nullptr, nullptr, 0, &key);
    if (rc < 0) return rc;
    int ii, jj, tt, dd;
    or_unpack(key, &ii, &jj, &tt, &dd);
    *i = ii;
    *j = jj;
    *type = tt;
    *delta = dd;
    return TSP2OPT_OK;
}
