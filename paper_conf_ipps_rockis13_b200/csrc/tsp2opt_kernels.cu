// tsp2opt_kernels.cu -- sm_100a kernels of the exhaustive best-improvement
// 2-opt hot path:
//   load_tour_kernel  a2 reorder P[k] = coords[tour[k]], P[n] = P[0]  + a3 edges e[k], length
//   sweep_kernel      a4 all pairs i < j of one (row-block x column-chunk) tile + a5 reduce
//   apply_kernel      a7 segment reversal, edges, length; a8 loop-control state
// Paper: L14 Alg. 2 (one job per pair, best value to global memory), L16 §IV.A
// (coordinates in on-chip memory, per-thread local best then global best),
// L18 §IV.B / L20 Fig. 7-8 (problem division into two coordinate sub-ranges,
// tiles over the upper triangle only).  Design and B200 rationale: DESIGN.md §5.
#include "tsp2opt_device.cuh"
#include "tsp2opt_internal.h"
#include "tsp2opt_sweep.cuh"

#include <type_traits>

namespace tsp2opt {

#ifdef TSP2OPT_PHASE_TIMING
// Instrumented builds only: clock cycles CTA 0 spends in each phase of the
// persistent incremental local search (boxes, barrier, sweep, barrier, apply,
// barrier), summed over the iterations; read by tsp2opt_debug_stats.
__device__ unsigned long long g_phase[16];
__device__ unsigned long long g_phase_it[8];  // per-iteration maxima, folded into g_phase[8..11] by CTA 0
#endif

// ===========================================================================
// a2 + a3: route-order gather and edge pass (L18 Fig. 6 "An array containing
// coordinates in the route's order"; done on the device instead of the host).
// Also validates the permutation (stamp array, one epoch per load).
// ===========================================================================
__global__ void __launch_bounds__(256) load_tour_kernel(const int* __restrict__ coords, const int* __restrict__ tour_src,
                                                        int* __restrict__ tour_dst, float2* __restrict__ P,
                                                        int* __restrict__ E, int n, Slot* __restrict__ slot,
                                                        unsigned* __restrict__ stamp, unsigned epoch)
{
    __shared__ long long red[8];
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    long long e = 0;
    if (k < n) {
        int c = tour_src[k];
        int c1 = tour_src[(k + 1 == n) ? 0 : k + 1];
        bool ok = (c >= 0 && c < n);
        if (ok) ok = atomicExch(&stamp[c], epoch) != epoch;  // a city seen twice -> not a permutation
        if (!ok) atomicOr(&slot->done, 4);
        if (c < 0 || c >= n) c = 0;
        if (c1 < 0 || c1 >= n) c1 = 0;
        const int xa = coords[2 * c], ya = coords[2 * c + 1];
        const int xb = coords[2 * c1], yb = coords[2 * c1 + 1];
        tour_dst[k] = c;
        const float2 p = make_float2(bias_coord(xa), bias_coord(ya));
        P[k] = p;
        if (k == 0) P[n] = p;  // closed array: position n is position 0 (reading R10)
        const int d = exact_dist_xy(xa, ya, xb, yb);
        E[k] = d;
        e = d;
    }
    for (int o = 16; o > 0; o >>= 1) e += __shfl_xor_sync(0xffffffffu, e, o);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = e;
    __syncthreads();
    if (threadIdx.x == 0) {
        long long s = 0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) s += red[w];
        atomicAdd((unsigned long long*)&slot->length, (unsigned long long)s);
    }
}

__global__ void init_slot_kernel(Slot* slot, int clear_length)
{
    slot->key = seed_key();
    slot->last_key = seed_key();
    slot->moves = 0;
    if (clear_length) slot->length = 0;
    slot->done = 0;
    slot->next_tile = 0;
    slot->ncull = 0;
    slot->seed_ok = 0;  // a freshly loaded tour: no previous sweep to seed from
    slot->mtype = 0;
}

// best_move's sweep is not followed by an apply: its tile minima must not be
// combined with an older move by a later sweep.
// ILS perturbation (L18 §V "a simple doublebridge move"): out = A C B D for
// in = A B C D, A = [0, a), B = [a, b), C = [b, c), D = [c, n); one thread per
// output position.
__global__ void double_bridge_kernel(const int* __restrict__ in, int* __restrict__ out, int n, int a, int b, int c)
{
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= n) return;
    int src;
    if (k < a || k >= c) src = k;                 // A and D stay
    else if (k < a + (c - b)) src = b + (k - a);  // C moves forward
    else src = a + (k - a - (c - b));             // B moves back
    out[k] = in[src];
}

__global__ void reset_key_kernel(Slot* slot)
{
    slot->key = seed_key();
    slot->seed_ok = 0;
}

// a4 + a5: the sweep of one tile lives in tsp2opt_sweep.cuh.
constexpr int kIncLsThreads = 512;     // persistent searches: 16 warps, one CTA per SM
constexpr int kIncLsMaxThreads = 512;
constexpr int kIncPartCols = 4;        // columns per part of a kept tile (inc_kept_parts)

#ifndef TSP2OPT_MINB
#define TSP2OPT_MINB 4  // CTAs of 128 threads per SM the register allocation must allow
#endif
template <int R, bool FIRST>
#ifndef TSP2OPT_SWEEP_LB_T
#define TSP2OPT_SWEEP_LB_T 128  // experiment: (32, 20) forces 102 registers for 20 one-warp CTAs per SM
#define TSP2OPT_SWEEP_LB_B TSP2OPT_MINB
#endif
#ifdef TSP2OPT_SWEEP_MAXNREG  // experiment: a register cap between the launch-bounds steps
#define TSP2OPT_SWEEP_ATTR __maxnreg__(TSP2OPT_SWEEP_MAXNREG)
#else
#define TSP2OPT_SWEEP_ATTR __launch_bounds__(TSP2OPT_SWEEP_LB_T, TSP2OPT_SWEEP_LB_B)
#endif
__global__ void TSP2OPT_SWEEP_ATTR sweep_kernel(const float2* __restrict__ P, const int* __restrict__ E, int n,
                                                     const int2* __restrict__ tiles, int TJ, Slot* __restrict__ slot,
                                                     int respect_done, unsigned long long* __restrict__ tilebest,
                                                     int flags)
{
    extern __shared__ float4 smem[];
    const TileSmem sm(smem, TJ, R * (int)blockDim.x);
    pdl_trigger();
    pdl_wait();
    if (respect_done && *(volatile int*)&slot->done) return;  // converged: iteration is a no-op
    // (the warp-tile form for one-warp CTAs -- compile-time warp index, 63-70 instead of
    // about 71 instructions per step -- measured 1 % slower here, r02_exp_sweep.jsonl)
    sweep_tile<R, false, FIRST>(P, E, n, tiles[blockIdx.x], TJ, slot, sm, tilebest + blockIdx.x, flags);
}

// ===========================================================================
// Culled sweep (TSP2OPT_OPT_TILE_BOUNDS = 2): the tile-level bound of
// tile_may_pass, evaluated for every tile BEFORE the sweep from per-block
// summaries, so the sweep launches only over the tiles that survive.  A
// spatially coherent tour (the later sweeps of a local search) keeps a few
// percent of the tiles; visiting the others only to skip them cost most of a
// sweep (60k one-warp CTAs at n = 85900).
//
// Exactness: a pair with delta < 0 has D(i,j) <= e_i - 1 or
// D(i+1,j+1) <= e_j - 1 (otherwise delta >= 0); D(a,b) <= t <=> s <= t^2 + t.
// Every city a pair of the tile touches (i, i+1 in the row block, j, j+1 in
// the column chunk) lies in the block's / chunk's box, so s >= gap^2 of the
// two boxes, and every edge it compares is <= max(emax_rows, emax_cols).  If
// gap^2 > T^2 + T with T = max emax - 1, no pair of the tile has delta < 0,
// and pairs with delta >= 0 never change the sweep's result (it is the min
// over improving pairs, else the seed (0, 1, 0); reading R7).  Integer
// arithmetic, no rounding.
// ===========================================================================
// One warp per summary: row block b = positions [b*TI, min(b*TI + TI, n-1))
// (cities up to the block end + 1), column chunk c = [c*TJ, min(c*TJ + TJ, n))
// (cities up to + 1; P[n] = P[0]).
// With G (2.5-opt, reading R19) the box also carries gneg = max(-g_k) over its
// positions: a node-insertion move with delta < 0 needs D(i+1, j) <= -1 - g
// for g = g_{i+1} or g_j (tsp2opt_sweep25.cu), so the cull threshold becomes
// max(emax, gneg) - 1 of the two boxes.
__global__ void __launch_bounds__(256) box_kernel(const float2* __restrict__ P, const int* __restrict__ E,
                                                  const int* __restrict__ G, int n, int TI, int nrb, int TJ, int ncc,
                                                  Box* __restrict__ rbox, Box* __restrict__ cbox,
                                                  Slot* __restrict__ slot, int respect_done, int incremental,
                                                  int halo)
{
    pdl_trigger();
    pdl_wait();
    // the slot's fields are read together (one L2 round trip; the kernel is latency bound)
    const int done = respect_done ? *(volatile const int*)&slot->done : 0;
    const int seed_ok = incremental ? *(volatile const int*)&slot->seed_ok : 0;
    const unsigned long long mv = incremental ? *(volatile const unsigned long long*)&slot->last_key : 0ull;
    // the cull and the list sweep that follow start from zeroed counters (a
    // best_move sweep leaves them set on the slot the next iteration reads)
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        slot->ncull = 0;
        slot->next_tile = 0;
    }
    if (done) return;
    // incremental: only the summaries of blocks the last applied move touched
    // (P changed on [i+1, j], E on [i, j]) are recomputed; the others stand
    int dlo = 0, dhi = n;
    if (seed_ok) {
        dlo = key_i(mv) - halo;  // halo 1 for 2.5-opt: the gains changed on [i, j+1]
        dhi = key_j(mv) + halo;
    }
    const int lane = threadIdx.x & 31;
    const int nwarps = (int)(gridDim.x * blockDim.x) >> 5;
    // grid-stride over the summaries: a small grid, most summaries are clean and skipped
    for (int w = (int)(blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nrb + ncc; w += nwarps) {
        int k0, ke;
        Box* out;
        if (w < nrb) {
            k0 = w * TI;
            ke = min(k0 + TI, n - 1);
            out = rbox + w;
        } else {
            k0 = (w - nrb) * TJ;
            ke = min(k0 + TJ, n);
            out = cbox + (w - nrb);
        }
        if (ke < dlo || k0 > dhi) continue;  // clean: its summary stands (whole warp)
        int xlo = 1 << 30, xhi = -1, ylo = 1 << 30, yhi = -1, emax = 0, gneg = 0;
        // up to kBoxIters positions per lane, all loads issued before the first use
        constexpr int kBoxIters = (32 * kRowsLarge * kMaxWarps + 1 + 31) / 32;
#pragma unroll
        for (int it = 0; it < kBoxIters; it++) {
            const int k = k0 + lane + 32 * it;
            if (k <= ke) {
                const float2 p = P[k];
                const int x = unbias(p.x), y = unbias(p.y);
                xlo = min(xlo, x);
                xhi = max(xhi, x);
                ylo = min(ylo, y);
                yhi = max(yhi, y);
                if (k < ke) emax = max(emax, E[k]);
                if (G) gneg = max(gneg, -G[k == n ? 0 : k]);
            }
        }
        const unsigned full = 0xffffffffu;
        xlo = __reduce_min_sync(full, xlo);
        xhi = __reduce_max_sync(full, xhi);
        ylo = __reduce_min_sync(full, ylo);
        yhi = __reduce_max_sync(full, yhi);
        emax = __reduce_max_sync(full, emax);
        gneg = __reduce_max_sync(full, gneg);
        if (lane == 0) {
            Box b;
            b.xlo = xlo;
            b.xhi = xhi;
            b.ylo = ylo;
            b.yhi = yhi;
            b.emax = emax;
            b.pad[0] = gneg;  // 0 without G
            b.pad[1] = b.pad[2] = 0;
            *out = b;
        }
    }
}

#ifndef TSP2OPT_CULL_V
#define TSP2OPT_CULL_V 4
#endif
#ifndef TSP2OPT_BOX_BLOCKS
#define TSP2OPT_BOX_BLOCKS 64  // box kernel grid cap (grid-stride over the summaries)
#endif
// One thread per tile of the shard: keep the tile iff its boxes allow a pair
// with delta < 0; kept tiles (I0, J0, index) are appended to list[] (warp-aggregated
// atomic on slot->ncull).  With seeding or the incremental sweep, a culled
// tile's minimum is "none".
constexpr int kCullPerThread = TSP2OPT_CULL_V;  // tiles per thread, their loads batched (the kernel is latency bound)

__global__ void __launch_bounds__(256) cull_kernel(const int2* __restrict__ tiles, int ntiles, int TI, int TJ,
                                                   const Box* __restrict__ rbox, const Box* __restrict__ cbox,
                                                   Slot* __restrict__ slot, int4* __restrict__ list,
                                                   unsigned long long* __restrict__ tilebest, int flags,
                                                   int respect_done, int n, int halo)
{
    constexpr int V = kCullPerThread;
    pdl_trigger();
    pdl_wait();
    // kSweepIncremental: a tile whose pairs (a, b) all have a, b outside the
    // last applied move's [i, j] is clean -- positions a, a+1, b, b+1 kept
    // their cities and e_a, e_b their lengths, so every delta and the tile's
    // stored minimum stand.  Otherwise (or without a valid last move) it is
    // culled (minimum: none) or listed for the sweep.
    // All independent loads first (the slot's fields, then V tiles per thread).
    const bool inc = (flags & kSweepIncremental) && !(flags & kSweepFull);
    const int done = respect_done ? *(volatile int*)&slot->done : 0;
    const int seed_ok = inc ? *(volatile int*)&slot->seed_ok : 0;
    const unsigned long long mv = inc ? *(volatile unsigned long long*)&slot->last_key : 0ull;
    const int gid = blockIdx.x * blockDim.x + threadIdx.x, stride = gridDim.x * blockDim.x;
    int2 tl[V];
    unsigned long long stored[V];
    bool live[V];
#pragma unroll
    for (int k = 0; k < V; k++) {
        const int t = gid + k * stride;
        live[k] = t < ntiles;
        tl[k] = make_int2(0, 0);
        stored[k] = kKeyNone;
        if (live[k]) {
            tl[k] = tiles[t];
            if (inc) stored[k] = tilebest[t];
        }
    }
    if (done) return;  // grid-uniform
    int dlo = 0, dhi = n;
    if (seed_ok) {
        dlo = key_i(mv) - halo;  // 2.5-opt (halo 1): a pair also reads g_{a+1}, g_b and D(a+1, b)
        dhi = key_j(mv) + halo;
    }
    unsigned long long clean_min = kKeyNone;
#pragma unroll
    for (int k = 0; k < V; k++)
        if (live[k]) {
            live[k] = (tl[k].x <= dhi && tl[k].x + TI >= dlo) || (tl[k].y <= dhi && tl[k].y + TJ >= dlo);  // dirty
            if (!live[k]) clean_min = min(clean_min, stored[k]);  // a clean tile's stored minimum stands
        }
    if (flags & kSweepIncremental) {
        // the clean tiles' share of the sweep's minimum (the re-swept tiles add
        // theirs from the list sweep); one atomic per block at most
        __shared__ unsigned long long s_min[8];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) clean_min = min(clean_min, __shfl_xor_sync(0xffffffffu, clean_min, o));
        if ((threadIdx.x & 31) == 0) s_min[threadIdx.x >> 5] = clean_min;
        __syncthreads();
        if (threadIdx.x == 0) {
            for (int w = 1; w < (int)(blockDim.x >> 5); w++) clean_min = min(clean_min, s_min[w]);
            if (clean_min != kKeyNone) atomicMin(&slot->key, clean_min);  // no read-back: a RED, no round trip
        }
    }
    Box r[V], c[V];
#pragma unroll
    for (int k = 0; k < V; k++)
        if (live[k]) {
            r[k] = rbox[tl[k].x / TI];
            c[k] = cbox[tl[k].y / TJ];
        }
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int k = 0; k < V; k++) {
        bool keep = false;
        if (live[k]) {
            const long long gx = max(0, max(c[k].xlo - r[k].xhi, r[k].xlo - c[k].xhi));
            const long long gy = max(0, max(c[k].ylo - r[k].yhi, r[k].ylo - c[k].yhi));
            const long long T =
                (long long)max(max(r[k].emax, c[k].emax), max(r[k].pad[0], c[k].pad[0])) - 1;  // pad[0]: gneg
            keep = T >= 0 && gx * gx + gy * gy <= T * T + T;
            if (!keep && (flags & (kSweepSeed | kSweepIncremental))) tilebest[gid + k * stride] = kKeyNone;
        }
        const unsigned m = __ballot_sync(0xffffffffu, keep);
        if (m) {
            const int leader = __ffs(m) - 1;
            unsigned base = 0;
            if (lane == leader) base = atomicAdd(&slot->ncull, (unsigned)__popc(m));
            base = __shfl_sync(0xffffffffu, base, leader);
            if (keep) list[base + __popc(m & ((1u << lane) - 1u))] = make_int4(tl[k].x, tl[k].y, gid + k * stride, 0);
        }
    }
}

// The sweep over the culled list: a grid of co-resident CTAs takes list
// entries one at a time -- entry blockIdx.x first, then claims from
// slot->next_tile (dynamic scheduling: the kept tiles of a coherent tour
// cluster along the diagonal, per-tile claims keep the CTAs balanced) until
// the list is done.
template <int R, bool FIRST>
__global__ void __launch_bounds__(128, TSP2OPT_MINB) sweep_list_kernel(const float2* __restrict__ P,
                                                                      const int* __restrict__ E, int n,
                                                                      const int2* __restrict__ tiles,
                                                                      const int4* __restrict__ list, int TJ,
                                                                      Slot* __restrict__ slot, int respect_done,
                                                                      unsigned long long* __restrict__ tilebest,
                                                                      int flags)
{
    extern __shared__ float4 smem[];
    const TileSmem sm(smem, TJ, R * (int)blockDim.x);
    __shared__ int4 s_t;
    pdl_trigger();
    pdl_wait();
    const int done = respect_done ? *(volatile int*)&slot->done : 0;  // both fields in one round trip
    const unsigned count = *(volatile unsigned*)&slot->ncull;
    if (done) return;
    // first entry static (entry blockIdx.x: no burst of 3k atomics on one
    // address at kernel start), then dynamic claims past the first wave
    unsigned k = blockIdx.x;
    for (;;) {
        if (threadIdx.x == 0) s_t = k < count ? list[k] : make_int4(0, 0, -1, 0);
        __syncthreads();
        const int4 e = s_t;
        if (e.z < 0) break;
        if (blockDim.x == 32)
            sweep_tile<R, false, FIRST, true>(P, E, n, make_int2(e.x, e.y), TJ, slot, sm, tilebest + e.z, flags);
        else
            sweep_tile<R, false, FIRST>(P, E, n, make_int2(e.x, e.y), TJ, slot, sm, tilebest + e.z, flags);
        if (threadIdx.x == 0) k = gridDim.x + atomicAdd(&slot->next_tile, 1u);
        __syncthreads();  // before the next tile overwrites the shared chunk (and s_t)
    }
}

// ===========================================================================
// Fused incremental culled sweep (TSP2OPT_OPT_TILE_BOUNDS = 3, every iteration
// after the first of a local search).  One launch replaces box + cull + list
// sweep: the dirty tiles -- those whose row block or column chunk meets the
// last applied move's [i, j] -- are ENUMERATED from (i, j) by index arithmetic
// (tmap: (row block, column chunk) -> this shard's tile index, -1 if none), not
// found by scanning all tiles; the warp that owns a dirty tile recomputes the
// boxes of its dirty blocks from P / E on the spot (no box kernel, no list),
// applies the cull test of cull_kernel and, if the tile is kept, sweeps it with
// its tile-local bound right away (kSweepLocal: the stored minimum stays exact
// while the tile is clean).  Every CTA also folds a share of the clean tiles'
// stored minima into the slot key.  Exactness: the same cull condition, the
// same tile sweep and the same clean / dirty rule as box_kernel + cull_kernel
// + sweep_list_kernel.
// ===========================================================================
__device__ __forceinline__ Box warp_box(const float2* P, const int* E, int k0, int ke)  // coherent loads: P, E may
                                                                                       // change within a launch
{
    // positions k0..ke (cities), edges k0..ke-1; every lane returns the box.  Up to
    // kWarpBoxBatch positions per lane have their loads issued before the first use
    // (one L2 round trip for a 225-position row block, instead of one per position).
    constexpr int kWarpBoxBatch = 8;
    int xlo = 1 << 30, xhi = -1, ylo = 1 << 30, yhi = -1, emax = 0;
    const int lane = threadIdx.x & 31;
    for (int k1 = k0; k1 <= ke; k1 += 32 * kWarpBoxBatch) {
        float2 p[kWarpBoxBatch];
        int e[kWarpBoxBatch];
#pragma unroll
        for (int b = 0; b < kWarpBoxBatch; b++) {
            const int k = k1 + lane + 32 * b;
            p[b] = k <= ke ? P[k] : make_float2(0.f, 0.f);
            e[b] = k < ke ? E[k] : 0;
        }
#pragma unroll
        for (int b = 0; b < kWarpBoxBatch; b++) {
            const int k = k1 + lane + 32 * b;
            if (k <= ke) {
                const int x = unbias(p[b].x), y = unbias(p[b].y);
                xlo = min(xlo, x);
                xhi = max(xhi, x);
                ylo = min(ylo, y);
                yhi = max(yhi, y);
                emax = max(emax, e[b]);
            }
        }
    }
    const unsigned full = 0xffffffffu;
    Box b;
    b.xlo = __reduce_min_sync(full, xlo);
    b.xhi = __reduce_max_sync(full, xhi);
    b.ylo = __reduce_min_sync(full, ylo);
    b.yhi = __reduce_max_sync(full, yhi);
    b.emax = __reduce_max_sync(full, emax);
    b.pad[0] = b.pad[1] = b.pad[2] = 0;
    return b;
}

template <int R, bool FIRST>
__global__ void __launch_bounds__(32, 16) inc_sweep_kernel(const float2* __restrict__ P, const int* __restrict__ E,
                                                           int n, const int2* __restrict__ tiles, int ntiles,
                                                           const int* __restrict__ tmap, int TI, int TJ, int nrb,
                                                           int ncc, Box* __restrict__ rbox, Box* __restrict__ cbox,
                                                           Slot* __restrict__ slot, int respect_done,
                                                           unsigned long long* __restrict__ tilebest, int flags)
{
    extern __shared__ float4 smem[];
    const TileSmem sm(smem, TJ, R * (int)blockDim.x);
    pdl_trigger();
    pdl_wait();
    const int done = respect_done ? *(volatile const int*)&slot->done : 0;
    const int seed_ok = *(volatile const int*)&slot->seed_ok;
    const unsigned long long mv = *(volatile const unsigned long long*)&slot->last_key;
    if (done) return;
    int dlo = 0, dhi = n;  // no valid last move: every tile is dirty
    if (seed_ok) {
        dlo = key_i(mv);
        dhi = key_j(mv);
    }
    const int lane = threadIdx.x & 31;
    // (1) the clean tiles' stored minima (a tile is clean iff neither its row
    //     range nor its column range meets [dlo, dhi]), one grid-stride pass
    {
        unsigned long long m = kKeyNone;
        constexpr int V = 4;  // loads in flight per lane
        for (int t0 = blockIdx.x * 32 * V; t0 < ntiles; t0 += gridDim.x * 32 * V) {
            int2 tl[V];
            unsigned long long kb[V];
#pragma unroll
            for (int v = 0; v < V; v++) {
                const int t = t0 + v * 32 + lane;
                tl[v] = t < ntiles ? tiles[t] : make_int2(0, 0);
                kb[v] = t < ntiles ? tilebest[t] : kKeyNone;
            }
#pragma unroll
            for (int v = 0; v < V; v++) {
                const bool dirty = (tl[v].x <= dhi && tl[v].x + TI >= dlo) || (tl[v].y <= dhi && tl[v].y + TJ >= dlo);
                if (!dirty) m = min(m, kb[v]);
            }
        }
        for (int o = 16; o > 0; o >>= 1) m = min(m, __shfl_xor_sync(0xffffffffu, m, o));
        if (lane == 0 && m != kKeyNone && m < *(volatile unsigned long long*)&slot->key) atomicMin(&slot->key, m);
    }
    // (2) the dirty tiles: rows [rlo, rhi] x every chunk, then every row block x
    //     chunks [clo, chi] without the rows already covered
    const int rlo = max(0, (dlo - TI + TI - 1) >= 0 ? (dlo - TI + TI - 1) / TI : 0), rhi = min(nrb - 1, dhi / TI);
    const int clo = max(0, (dlo - TJ + TJ - 1) >= 0 ? (dlo - TJ + TJ - 1) / TJ : 0), chi = min(ncc - 1, dhi / TJ);
    const long long nA = rlo <= rhi ? (long long)(rhi - rlo + 1) * ncc : 0;
    const long long nB = clo <= chi ? (long long)nrb * (chi - clo + 1) : 0;
    for (long long u = blockIdx.x; u < nA + nB; u += gridDim.x) {
        int rb, cc;
        if (u < nA) {
            rb = rlo + (int)(u / ncc);
            cc = (int)(u % ncc);
        } else {
            const long long v = u - nA;
            rb = (int)(v / (chi - clo + 1));
            cc = clo + (int)(v % (chi - clo + 1));
            if (rb >= rlo && rb <= rhi) continue;  // already in part A
        }
        const int t = tmap[(long long)rb * ncc + cc];
        if (t < 0) continue;  // below the diagonal, or another rank's tile
        const bool rdirty = rb >= rlo && rb <= rhi, cdirty = cc >= clo && cc <= chi;
        Box r, c;
        if (rdirty) {
            r = warp_box(P, E, rb * TI, min(rb * TI + TI, n - 1));
            if (lane == 0) rbox[rb] = r;  // every warp of this row writes the same box
        } else {
            r = rbox[rb];
        }
        if (cdirty) {
            c = warp_box(P, E, cc * TJ, min(cc * TJ + TJ, n));
            if (lane == 0) cbox[cc] = c;
        } else {
            c = cbox[cc];
        }
        const long long gx = max(0, max(c.xlo - r.xhi, r.xlo - c.xhi));
        const long long gy = max(0, max(c.ylo - r.yhi, r.ylo - c.yhi));
        const long long T = (long long)max(r.emax, c.emax) - 1;
        const bool keep = T >= 0 && gx * gx + gy * gy <= T * T + T;
        if (keep) {
            sweep_tile<R, false, FIRST, true>(P, E, n, make_int2(rb * TI, cc * TJ), TJ, slot, sm, tilebest + t,
                                        flags | kSweepLocal);
            __syncthreads();  // before the next tile overwrites the shared chunk
        } else if (lane == 0) {
            tilebest[t] = kKeyNone;
        }
    }
}

template <int R, bool FIRST>
static cudaError_t launch_inc_sweep_t(const Geometry& g, const float2* P, const int* E, int n, const int2* tiles,
                                      int ntiles, const int* tmap, int grid, Box* rbox, Box* cbox, Slot* slot,
                                      int respect_done, unsigned long long* tilebest, int flags, cudaStream_t st)
{
    const int TI = g.ti(), nrb = (n - 1 + TI - 1) / TI, ncc = (n + g.tj - 1) / g.tj;
    return launch_kernel_pdl(inc_sweep_kernel<R, FIRST>, dim3(grid), dim3(32), sweep_smem_bytes(g), st, P, E, n,
                             tiles, ntiles, tmap, TI, g.tj, nrb, ncc, rbox, cbox, slot, respect_done, tilebest,
                             flags & ~kSweepSeed);
}

// ===========================================================================
// a7 + a8: apply the best move of slot_in (or an explicit (i, j)) and write
// the next iteration's state into slot_out.  Reverses P and tour on [i+1, j]
// and e on [i+1, j-1]; the two new edges are exact distances of the
// pre-reversal cities (thread 0 reads them before doing its own swap; no other
// thread touches P[i], P[i+1], P[j], P[j+1], e[i], e[j]).
// ===========================================================================
// Returns whether a move was applied (false: converged / capped / already done).
__device__ __forceinline__ bool apply_phase(float2* __restrict__ P, int* __restrict__ E, int* __restrict__ tour,
                                            const Slot* __restrict__ in, Slot* __restrict__ out, long long max_moves,
                                            int explicit_move, int ei, int ej, int gtid, int stride,
                                            unsigned long long* __restrict__ trace, long long trace_cap,
                                            int* __restrict__ pos)
{
    const unsigned long long key = in->key;
    const int done = in->done;
    const long long moves = in->moves;
    int i, j;
    bool apply;
    if (explicit_move) {
        i = ei;
        j = ej;
        apply = true;
    } else {
        i = key_i(key);
        j = key_j(key);
        apply = !done && key_delta(key) < 0 && moves < max_moves;
    }
    if (gtid == 0) {
        Slot o;
        o.key = seed_key();
        o.last_key = explicit_move ? in->last_key : key;
        o.moves = moves;
        o.length = in->length;
        o.done = explicit_move ? (done & 4) : done;  // an explicit move makes the tour unconverged
        o.next_tile = 0;
        o.ncull = 0;
        o.mtype = 0;
        o.seed_ok = (apply && !explicit_move) ? 1 : 0;  // tile minima of this sweep seed the next one
        if (!explicit_move && !done) {
            if (key_delta(key) >= 0) o.done = 1;        // local minimum (reading R7)
            else if (moves >= max_moves) o.done = 2;    // capped with an improving move left (R8)
        }
        if (apply) {
            // thread 0 alone swaps positions i+1 <-> j and writes E[i], E[j], so these reads
            // see the pre-move state even while other threads (and CTAs) reverse the rest
            const float2 pi = __ldcg(P + i), pj = __ldcg(P + j), pi1 = __ldcg(P + i + 1), pj1 = __ldcg(P + j + 1);
            const int ni = exact_dist_biased(pi, pj), nj = exact_dist_biased(pi1, pj1);
            const int d = ni + nj - __ldcg(E + i) - __ldcg(E + j);
            o.length += d;
            o.moves = moves + 1;
            E[i] = ni;
            E[j] = nj;
            if (!explicit_move) {
                // the applied move with its exact delta: a first-improvement key carries the
                // marker delta (reading R20) until here; a best-improvement key already has d
                o.last_key = pack_key(d, i, j);
                if (trace && moves < trace_cap) trace[moves] = o.last_key;  // move trace (tests)
            }
        }
        *out = o;
    }
    if (!apply) return false;
    const int half = (j - i) >> 1;  // swap P/tour positions i+1+t <-> j-t
    for (int t = gtid; t < half; t += stride) {
        const int a = i + 1 + t, c = j - t;
        const float2 pa = __ldcg(P + a), pc = __ldcg(P + c);
        P[a] = pc;
        P[c] = pa;
        const int ta = __ldcg(tour + a), tc = __ldcg(tour + c);
        tour[a] = tc;
        tour[c] = ta;
        if (pos) {  // pruned sweep: keep the inverse permutation current
            pos[tc] = a;
            pos[ta] = c;
        }
    }
    const int ehalf = (j - i - 1) >> 1;  // swap e positions i+1+t <-> j-1-t
    for (int t = gtid; t < ehalf; t += stride) {
        const int a = i + 1 + t, c = j - 1 - t;
        const int ea = __ldcg(E + a), ec = __ldcg(E + c);
        E[a] = ec;
        E[c] = ea;
    }
    return true;
}

__global__ void __launch_bounds__(256) apply_kernel(float2* __restrict__ P, int* __restrict__ E, int* __restrict__ tour,
                                                    const Slot* __restrict__ in, Slot* __restrict__ out,
                                                    long long max_moves, int explicit_move, int ei, int ej,
                                                    unsigned long long* __restrict__ trace, long long trace_cap,
                                            int* __restrict__ pos)
{
    __shared__ Slot s_in;  // one read of the input state per block
    pdl_trigger();
    pdl_wait();
    if (threadIdx.x == 0) s_in = *in;
    __syncthreads();
    apply_phase(P, E, tour, &s_in, out, max_moves, explicit_move, ei, ej, blockIdx.x * blockDim.x + threadIdx.x,
                gridDim.x * blockDim.x, trace, trace_cap, pos);
}

// ===========================================================================
// Device-resident local search (§8(a) a4-a8 in ONE launch, world == 1): a
// persistent cooperative grid alternates {sweep over all tiles, dynamically
// scheduled; grid barrier; apply; grid barrier} until the local minimum, the
// move cap or the per-launch iteration budget.  Slots ping-pong exactly as in
// the multi-kernel path; the final parity is written to ctl[0].
// ===========================================================================
// grid_sync: tsp2opt_device.cuh

template <int R>
__global__ void __launch_bounds__(128, TSP2OPT_MINB) local_search_kernel(float2* __restrict__ P, int* __restrict__ E,
                                                           int* __restrict__ tour, int n,
                                                           const int2* __restrict__ tiles, int ntiles, int TJ,
                                                           Slot* __restrict__ slots, int parity, long long max_moves,
                                                           long long budget, unsigned* __restrict__ bar,
                                                           int* __restrict__ ctl,
                                                           unsigned long long* __restrict__ tilebest, int flags,
                                                           unsigned long long* __restrict__ trace, long long trace_cap)
{
    extern __shared__ float4 smem[];
    const TileSmem sm(smem, TJ, R * (int)blockDim.x);
    __shared__ Slot s_in;
    const int gtid = blockIdx.x * blockDim.x + threadIdx.x;
    const int stride = gridDim.x * blockDim.x;
    int p = parity;
    unsigned long long target = 0;  // monotonic barrier on bar (reset to 0 before the launch)
    unsigned long long* ctr = reinterpret_cast<unsigned long long*>(bar);
    for (long long it = 0; it < budget; it++) {
        Slot* in = slots + p;
        // one read of the settled state per block (not one per thread: a single hot address)
        if (threadIdx.x == 0) s_in.done = *(volatile int*)&in->done;
        __syncthreads();
        if (s_in.done) break;  // uniform across the grid
        // a4/a5: tiles are assigned round-robin (largest first); the grid is co-resident
        for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
            sweep_tile<R, true>(P, E, n, tiles[t], TJ, in, sm, tilebest + t, flags);
            __syncthreads();  // before the next tile overwrites the shared chunk
        }
        grid_sync_mono(ctr, target);
        if (threadIdx.x == 0) {
            s_in.key = *(volatile unsigned long long*)&in->key;
            s_in.last_key = in->last_key;
            s_in.moves = *(volatile long long*)&in->moves;
            s_in.length = *(volatile long long*)&in->length;
            s_in.done = *(volatile int*)&in->done;
            s_in.seed_ok = *(volatile int*)&in->seed_ok;
        }
        __syncthreads();
        apply_phase(P, E, tour, &s_in, slots + (p ^ 1), max_moves, 0, 0, 0, gtid, stride, trace, trace_cap, nullptr);
        p ^= 1;
        grid_sync_mono(ctr, target);
    }
    if (gtid == 0) ctl[0] = p;
}

// Phase (C2) of the persistent incremental search with kept tiles split into
// column parts: the CTA's threads cull the dirty tiles enumerated CTA-major
// (u = thread * grid + CTA, so the clustered kept tiles of one move spread over
// the CTAs; the tile index, both boxes loaded in one round trip), collect the
// kept ones in a shared list, stage up to kStageTiles of them at once (every
// thread loads; one L2 round trip) and the CTA's warps sweep (tile, part)
// items with sweep_part; the tile minimum is the shared atomicMin over its
// parts.  Same cull test, tile-local bound and stored minima as the per-warp
// tile sweep, so the same moves.  Minima go to tilebest[t] (tb2 == nullptr) or,
// for inc_ls2_kernel, to the dense per-(row block, column chunk) array tb2
// plus an atomicMin into the tile's group minimum sm2 (64 chunks per group).
constexpr int kStageTiles = 16;
constexpr int kGroupChunks = 64;  // column chunks per group minimum (inc_ls2_kernel)
template <int R, bool FIRST>
__device__ __forceinline__ void inc_kept_parts(const float2* P, const int* E, int n,
                                               const int* __restrict__ tmap, int TI, int TJ, int nrb, int ncc,
                                               int rlo, int rhi, int clo, int chi, long long nA, long long nB,
                                               const Box* rbox, const Box* cbox,
                                               Slot* in, unsigned long long* tilebest,
                                               int tflags, int part_cols, float4* smem, int tile_bytes,
                                               unsigned long long* tb2 = nullptr, unsigned long long* sm2 = nullptr,
                                               int nsc = 0)
{
    __shared__ int s_nk;
    __shared__ int4 s_kt[kIncLsMaxThreads];  // kept tiles of this round: (t, rb, cc)
    __shared__ unsigned long long s_tmin[kStageTiles];
    const int tid = threadIdx.x, nthr = blockDim.x, wib = tid >> 5, nwb = nthr >> 5;
    const int nparts = (TJ + part_cols - 1) / part_cols;
    const long long step = (long long)nthr * gridDim.x;
#ifdef TSP2OPT_PHASE_TIMING
    // per CTA: [2] cull cycles, [3] staging, [4] part sweeps, [5] kept tiles -- maxima over CTAs per move
    long long pt0 = clock64(), pcull = 0, pstage = 0, pitems = 0;
    int pkept = 0;
#endif
    for (long long base = 0; base < nA + nB; base += step) {
        if (tid == 0) s_nk = 0;
        __syncthreads();
        const long long u = base + (long long)tid * gridDim.x + blockIdx.x;
        if (u < nA + nB) {
            int rb, cc;
            bool cand = true;
            if (u < nA) {
                rb = rlo + (int)(u / ncc);
                cc = (int)(u % ncc);
            } else {
                const long long v = u - nA;
                rb = (int)(v / (chi - clo + 1));
                cc = clo + (int)(v % (chi - clo + 1));
                cand = rb < rlo || rb > rhi;  // else already in part A
            }
            if (cand) {
                const int t = tmap[(long long)rb * ncc + cc];  // issued together with the two boxes
                const Box r = rbox[rb], c = cbox[cc];
                if (t >= 0) {
                    const long long gx = max(0, max(c.xlo - r.xhi, r.xlo - c.xhi));
                    const long long gy = max(0, max(c.ylo - r.yhi, r.ylo - c.yhi));
                    const long long T = (long long)max(r.emax, c.emax) - 1;
                    if (T >= 0 && gx * gx + gy * gy <= T * T + T) s_kt[atomicAdd(&s_nk, 1)] = make_int4(t, rb, cc, 0);
                    else if (tb2) tb2[(long long)rb * ncc + cc] = kKeyNone;
                    else tilebest[t] = kKeyNone;
                }
            }
        }
        __syncthreads();
        const int nk = s_nk;
#ifdef TSP2OPT_PHASE_TIMING
        {
            const long long t1 = clock64();
            pcull += t1 - pt0;
            pt0 = t1;
            pkept += nk;
        }
#endif
        for (int b0 = 0; b0 < nk; b0 += kStageTiles) {
            const int nb = min(kStageTiles, nk - b0);
            // stage: per tile the column positions J0 .. J1 + 1 and the row positions I0 .. I0 + 32R
            // (P and E of each), loads batched ahead of the shared stores
            const int ncolp = TJ + 2, nrowp = 32 * R + 1, per = ncolp + nrowp;
            constexpr int U = 8;
            for (int x0 = 0; x0 < nb * per; x0 += U * nthr) {
                float2 pv[U];
                int ev[U];
#pragma unroll
                for (int v = 0; v < U; v++) {
                    const int x = x0 + v * nthr + tid;
                    pv[v] = make_float2(0.f, 0.f);
                    ev[v] = 0;
                    if (x < nb * per) {
                        const int k = x / per, q = x - k * per;
                        const int4 kt = s_kt[b0 + k];
                        const int pos = q < ncolp ? kt.z * TJ + q : kt.y * TI + (q - ncolp);
                        pv[v] = P[pos];
                        ev[v] = E[pos];
                    }
                }
#pragma unroll
                for (int v = 0; v < U; v++) {
                    const int x = x0 + v * nthr + tid;
                    if (x < nb * per) {
                        const int k = x / per, q = x - k * per;
                        const TileSmem tsm(reinterpret_cast<char*>(smem) + (size_t)k * tile_bytes, TJ, 32 * R);
                        if (q < ncolp) {
                            tsm.put(q, pv[v], (float)ev[v]);
                        } else {
                            const int rq = q - ncolp;  // row position I0 + rq: lane rq / R, slot rq % R
                            const int ln = rq / R, sl = rq - ln * R;
                            if (ln < 32) {
                                tsm.rowp[ln * (R + 1) + sl] = pv[v];
                                tsm.rowe[rq] = (float)ev[v];
                            }
                            if (sl == 0 && ln > 0) tsm.rowp[(ln - 1) * (R + 1) + R] = pv[v];  // previous lane's row R
                        }
                    }
                }
            }
            if (tid < nb) s_tmin[tid] = kKeyNone;
            __syncthreads();
#ifdef TSP2OPT_PHASE_TIMING
            {
                const long long t1 = clock64();
                pstage += t1 - pt0;
                pt0 = t1;
            }
#endif
            for (int it = wib; it < nb * nparts; it += nwb) {
                const int k = it / nparts, part = it - k * nparts;
                const int4 kt = s_kt[b0 + k];
                const TileSmem tsm(reinterpret_cast<char*>(smem) + (size_t)k * tile_bytes, TJ, 32 * R);
                const int I0 = kt.y * TI, J0 = kt.z * TJ, J1 = min(J0 + TJ, n);
                const int jb = J0 + part * part_cols, je = min(jb + part_cols, J1);
                if (jb < je) {
                    const unsigned long long mk = sweep_part<R, FIRST>(I0, J0, jb, je, tsm, tflags);
                    if (mk != kKeyNone) atomicMin(&s_tmin[k], mk);
                }
            }
            __syncthreads();
#ifdef TSP2OPT_PHASE_TIMING
            {
                const long long t1 = clock64();
                pitems += t1 - pt0;
                pt0 = t1;
            }
#endif
            if (tid < nb) {
                const unsigned long long m = s_tmin[tid];
                const int4 kt = s_kt[b0 + tid];
                if (tb2) {
                    tb2[(long long)kt.y * ncc + kt.z] = m;
                    if (m != kKeyNone) atomicMin(&sm2[(long long)kt.y * nsc + kt.z / kGroupChunks], m);
                } else {
                    tilebest[kt.x] = m;
                }
                if (m != kKeyNone && m < *(volatile unsigned long long*)&in->key) atomicMin(&in->key, m);
            }
            __syncthreads();  // before the next batch restages the shared tiles
        }
    }
#ifdef TSP2OPT_PHASE_TIMING
    if (tid == 0) {
        atomicMax(&g_phase_it[2], (unsigned long long)pcull);
        atomicMax(&g_phase_it[3], (unsigned long long)pstage);
        atomicMax(&g_phase_it[4], (unsigned long long)pitems);
        atomicMax(&g_phase_it[5], (unsigned long long)pkept);
    }
#endif
}

// ===========================================================================
// Persistent incremental local search (TSP2OPT_OPT_TILE_BOUNDS = 3, one GPU):
// ONE cooperative launch runs the whole culled, incremental search of §5.6 --
// per iteration
//   (B) the boxes of the row blocks / column chunks the last move touched
//       (one warp each),                                          grid barrier,
//   (C) the clean tiles' stored minima folded into the key (every thread),
//       the dirty tiles culled (one THREAD each, enumerated from the last move
//       through tmap) and every kept tile swept by one WARP with its private
//       shared memory and the tile-local bound (kSweepLocal),    grid barrier,
//   (A) the apply of the winning move (apply_phase, every thread), grid barrier
// -- instead of four launches per move.  Same boxes, cull test, tile sweep,
// clean / dirty rule and apply as box_kernel + cull_kernel + sweep_list_kernel
// + apply_kernel, so the result is the same move sequence.  A dirty tile's
// lane index is warp-major (u = lane * warps + warp), so the kept tiles of
// one move -- neighbours in u -- land on different warps.  The first iteration
// of a launch with `full` set (or any without a valid last move) treats every
// block and tile as dirty: the full culled sweep.
// ===========================================================================
template <int R, bool FIRST>
__global__ void __launch_bounds__(512, 1) inc_ls_kernel(float2* __restrict__ P, int* __restrict__ E,
                                                        int* __restrict__ tour, int n,
                                                        const int2* __restrict__ tiles, int ntiles,
                                                        const int* __restrict__ tmap, int TI, int TJ, int nrb,
                                                        int ncc, Box* __restrict__ rbox, Box* __restrict__ cbox,
                                                        Slot* __restrict__ slots, int parity, long long max_moves,
                                                        long long budget, int full, unsigned* __restrict__ bar,
                                                        int* __restrict__ ctl,
                                                        unsigned long long* __restrict__ tilebest, int flags,
                                                        unsigned long long* __restrict__ trace, long long trace_cap,
                                                        int tile_bytes, int part_cols)
{
    extern __shared__ float4 smem[];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const TileSmem sm(reinterpret_cast<char*>(smem) + (size_t)wib * tile_bytes, TJ, 32 * R);  // this warp's tile memory
    const int nwb = blockDim.x >> 5;
    const int gw = blockIdx.x * nwb + wib, nw = gridDim.x * nwb;
    const int gtid = blockIdx.x * blockDim.x + threadIdx.x, stride = gridDim.x * blockDim.x;
    const int tflags = (flags | kSweepLocal) & ~kSweepSeed;
    __shared__ Slot s_in;
    __shared__ unsigned long long s_min[16];
    int p = parity;
#ifdef TSP2OPT_PHASE_TIMING
    long long tp0 = clock64();
#define PHASE_MARK(k)                                                                         \
    do {                                                                                      \
        if (blockIdx.x == 0 && threadIdx.x == 0) {                                            \
            const long long tp1 = clock64();                                                  \
            atomicAdd(&g_phase[k], (unsigned long long)(tp1 - tp0));                          \
            tp0 = tp1;                                                                        \
        }                                                                                     \
    } while (0)
#else
#define PHASE_MARK(k) \
    do {              \
    } while (0)
#endif
    for (long long it = 0; it < budget; it++) {
        Slot* in = slots + p;
        if (threadIdx.x == 0) {
            s_in.done = *(volatile int*)&in->done;
            s_in.seed_ok = (full && it == 0) ? 0 : *(volatile int*)&in->seed_ok;
            s_in.last_key = *(volatile unsigned long long*)&in->last_key;
        }
        __syncthreads();
        if (s_in.done) break;  // uniform across the grid
        int dlo = 0, dhi = n;
        if (s_in.seed_ok) {
            dlo = key_i(s_in.last_key);
            dhi = key_j(s_in.last_key);
        }
        const int rlo = dlo >= 1 ? (dlo - 1) / TI : 0, rhi = min(nrb - 1, dhi / TI);
        const int clo = dlo >= 1 ? (dlo - 1) / TJ : 0, chi = min(ncc - 1, dhi / TJ);
        // (B) boxes of the dirty blocks
        {
            const int nR = rhi - rlo + 1, nC = chi - clo + 1;
            for (int task = gw; task < nR + nC; task += nw) {
                if (task < nR) {
                    const int rb = rlo + task;
                    const Box b = warp_box(P, E, rb * TI, min(rb * TI + TI, n - 1));
                    if (lane == 0) rbox[rb] = b;
                } else {
                    const int cc = clo + task - nR;
                    const Box b = warp_box(P, E, cc * TJ, min(cc * TJ + TJ, n));
                    if (lane == 0) cbox[cc] = b;
                }
            }
        }
        PHASE_MARK(0);
        grid_sync(bar, gridDim.x);
        PHASE_MARK(1);
        // (C2) the dirty tiles: cull per thread, sweep the kept ones per warp
#ifdef TSP2OPT_PHASE_TIMING
        const long long tw0 = clock64();
        long long tcull = 0, tsweep = 0;
        int nkept = 0;
#endif
        const long long nA = (long long)(rhi - rlo + 1) * ncc;
        const long long nB = (long long)nrb * (chi - clo + 1);
        if (part_cols > 0) {
            inc_kept_parts<R, FIRST>(P, E, n, tmap, TI, TJ, nrb, ncc, rlo, rhi, clo, chi, nA, nB, rbox, cbox, in,
                                     tilebest, tflags, part_cols, smem, tile_bytes);
        } else
        for (long long base = 0; base < nA + nB; base += (long long)nw * 32) {
            const long long u = base + (long long)lane * nw + gw;
            int t = -1, rb = 0, cc = 0;
            if (u < nA + nB) {
                if (u < nA) {
                    rb = rlo + (int)(u / ncc);
                    cc = (int)(u % ncc);
                } else {
                    const long long v = u - nA;
                    rb = (int)(v / (chi - clo + 1));
                    cc = clo + (int)(v % (chi - clo + 1));
                }
                if (u < nA || rb < rlo || rb > rhi) t = tmap[(long long)rb * ncc + cc];
            }
            bool keep = false;
            if (t >= 0) {
                const Box r = rbox[rb], c = cbox[cc];
                const long long gx = max(0, max(c.xlo - r.xhi, r.xlo - c.xhi));
                const long long gy = max(0, max(c.ylo - r.yhi, r.ylo - c.yhi));
                const long long T = (long long)max(r.emax, c.emax) - 1;
                keep = T >= 0 && gx * gx + gy * gy <= T * T + T;
                if (!keep) tilebest[t] = kKeyNone;
            }
            unsigned kept = __ballot_sync(0xffffffffu, keep);
#ifdef TSP2OPT_PHASE_TIMING
            if (base == 0) tcull = clock64() - tw0;  // the first round's cull
            nkept += __popc(kept);
            const long long ts0 = clock64();
#endif
            while (kept) {  // this warp sweeps the kept tiles its lanes found
                const int src = __ffs(kept) - 1;
                kept &= kept - 1;
                const int kt = __shfl_sync(0xffffffffu, t, src);
                const int krb = __shfl_sync(0xffffffffu, rb, src), kcc = __shfl_sync(0xffffffffu, cc, src);
                sweep_tile<R, true, FIRST, true>(P, E, n, make_int2(krb * TI, kcc * TJ), TJ, in, sm, tilebest + kt,
                                                 tflags);
            }
#ifdef TSP2OPT_PHASE_TIMING
            tsweep += clock64() - ts0;
#endif
        }
#ifdef TSP2OPT_PHASE_TIMING
        if (lane == 0) {
            atomicMax(&g_phase_it[0], (unsigned long long)(clock64() - tw0));
            atomicMax(&g_phase_it[1], (unsigned long long)tsweep);
            atomicMax(&g_phase_it[2], (unsigned long long)tcull);
            atomicAdd(&g_phase_it[3], (unsigned long long)nkept);
        }
#endif
        PHASE_MARK(2);
        // (C1) the clean tiles' stored minima -- after the sweeps, so that warps
        // without kept tiles do it while the others still sweep; loads batched
        unsigned long long m = kKeyNone;
        if (s_in.seed_ok) {
            constexpr int V = 4;
            for (int t0 = gtid; t0 < ntiles; t0 += V * stride) {
                int2 tl[V];
                unsigned long long kb[V];
#pragma unroll
                for (int v = 0; v < V; v++) {
                    const int t = t0 + v * stride;
                    tl[v] = t < ntiles ? tiles[t] : make_int2(-(1 << 30), -(1 << 30));
                    kb[v] = t < ntiles ? tilebest[t] : kKeyNone;
                }
#pragma unroll
                for (int v = 0; v < V; v++) {
                    const bool dirty =
                        (tl[v].x <= dhi && tl[v].x + TI >= dlo) || (tl[v].y <= dhi && tl[v].y + TJ >= dlo);
                    if (!dirty) m = min(m, kb[v]);
                }
            }
        }
        for (int o = 16; o > 0; o >>= 1) m = min(m, __shfl_xor_sync(0xffffffffu, m, o));
        if (lane == 0) s_min[wib] = m;
        PHASE_MARK(6);
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned long long bm = s_min[0];
            for (int w = 1; w < nwb; w++) bm = min(bm, s_min[w]);
            if (bm != kKeyNone) atomicMin(&in->key, bm);
        }
        grid_sync(bar, gridDim.x);
        PHASE_MARK(3);
#ifdef TSP2OPT_PHASE_TIMING
        if (blockIdx.x == 0 && threadIdx.x == 0)
            for (int q = 0; q < 4; q++) {
                g_phase[8 + q] += g_phase_it[q];
                g_phase_it[q] = 0;
            }
#endif
        // (A) apply the winning move
        if (threadIdx.x == 0) {
            // first improvement: the key keeps its marker delta (< 0, so every CTA applies);
            // apply_phase's thread 0 derives the exact delta before its own swap (reading R20)
            s_in.key = *(volatile unsigned long long*)&in->key;
            s_in.moves = *(volatile long long*)&in->moves;
            s_in.length = *(volatile long long*)&in->length;
        }
        __syncthreads();
        apply_phase(P, E, tour, &s_in, slots + (p ^ 1), max_moves, 0, 0, 0, gtid, stride, trace, trace_cap, nullptr);
        p ^= 1;
        PHASE_MARK(4);
        grid_sync(bar, gridDim.x);
        PHASE_MARK(5);
    }
    if (gtid == 0) ctl[0] = p;
#undef PHASE_MARK
}

// ===========================================================================
// Persistent incremental local search, two grid barriers per move
// (inc_ls2_kernel; the default for TSP2OPT_OPT_TILE_BOUNDS = 3 on one GPU).
// Per move:
//   (C) the dirty tiles culled and the kept ones swept in column parts
//       (inc_kept_parts)                                          grid barrier,
//   (X) the move applied OUT OF PLACE -- the next state is written into the
//       other of two P / E / tour buffers, read only from the current one --
//       so that, in the same phase, the boxes of the blocks the move dirties
//       are computed from the current buffer through the reversal's mirror map
//       (new P[k] = P[i+j+1-k] on [i+1, j], new e[k] = e[i+j-k] on (i, j),
//       the two new edges), and the clean tiles' stored minima are folded into
//       the next sweep's key;                                      grid barrier.
// The buffer written by a move holds the state two moves back, so it is
// brought up to date on the previous move's positions and written on this
// move's (a few hundred entries for a typical move).  The launch starts with
// a full copy current -> alternate and ends by copying the last move's
// positions back if the current state is in the alternate buffer, so the
// handle's P / E / tour are current between launches.
// Clean minima: tile minima live in a dense (row block, column chunk) array
// tb2 and, per group of kGroupChunks chunks of one row block, in sm2 = the
// min over the group's tiles.  (X) resets sm2 of the groups the move dirties
// to the min over their clean tiles (none for a dirty row block) and (C)
// atomicMins every re-swept tile into its group, so sm2 is exact after every
// sweep; the clean scan reads one sm2 entry per clean group and the clean
// tiles of the (at most two) partly dirty groups of each row block, instead of
// every tile.  Same boxes, cull test, tile sweep, clean / dirty rule and
// decisions as the three-barrier kernel (inc_ls_kernel): the same moves.
// ===========================================================================
// Box of positions k0..ke (cities) and edges k0..ke-1 of the state AFTER move
// (i, j) (i < 0: no move), read from the state before it: city at k is
// P[i+j+1-k] on [i+1, j]; edge k is di / dj at i / j, e[i+j-k] on (i, j).
// di / dj are computed here from loads issued with the box's own.
__device__ __forceinline__ Box warp_box_mirror(const float2* P, const int* E, int k0, int ke, int i, int j)
{
    constexpr int kWarpBoxBatch = 8;
    const int lane = threadIdx.x & 31;
    float2 pi = make_float2(0.f, 0.f), pj = pi, pi1 = pi, pj1 = pi;
    const bool has_i = i >= k0 && i < ke, has_j = j >= k0 && j < ke;  // the new edges fall in this range
    if (has_i || has_j) {
        pi = P[i];
        pj = P[j];
        pi1 = P[i + 1];
        pj1 = P[j + 1];
    }
    int xlo = 1 << 30, xhi = -1, ylo = 1 << 30, yhi = -1, emax = 0;
    for (int k1 = k0; k1 <= ke; k1 += 32 * kWarpBoxBatch) {
        float2 p[kWarpBoxBatch];
        int e[kWarpBoxBatch];
#pragma unroll
        for (int b = 0; b < kWarpBoxBatch; b++) {
            const int k = k1 + lane + 32 * b;
            const int mk = (k > i && k <= j) ? i + j + 1 - k : k;
            const int me = (k > i && k < j) ? i + j - k : k;
            p[b] = k <= ke ? P[mk] : make_float2(0.f, 0.f);
            e[b] = (k < ke && k != i && k != j) ? E[me] : 0;
        }
#pragma unroll
        for (int b = 0; b < kWarpBoxBatch; b++) {
            const int k = k1 + lane + 32 * b;
            if (k <= ke) {
                const int x = unbias(p[b].x), y = unbias(p[b].y);
                xlo = min(xlo, x);
                xhi = max(xhi, x);
                ylo = min(ylo, y);
                yhi = max(yhi, y);
                emax = max(emax, e[b]);
            }
        }
    }
    if (has_i) emax = max(emax, exact_dist_biased(pi, pj));
    if (has_j) emax = max(emax, exact_dist_biased(pi1, pj1));
    const unsigned full = 0xffffffffu;
    Box b;
    b.xlo = __reduce_min_sync(full, xlo);
    b.xhi = __reduce_max_sync(full, xhi);
    b.ylo = __reduce_min_sync(full, ylo);
    b.yhi = __reduce_max_sync(full, yhi);
    b.emax = __reduce_max_sync(full, emax);
    b.pad[0] = b.pad[1] = b.pad[2] = 0;
    return b;
}

// Boxes of the blocks dirtied by move (i, j) over positions [dlo, dhi] (i < 0:
// no mirror, plain reads), one warp per block, warps gw of nw.
__device__ __forceinline__ void dirty_boxes(const float2* P, const int* E, int n, int TI, int TJ, int nrb, int ncc,
                                            int dlo, int dhi, int i, int j, Box* rbox, Box* cbox, int gw, int nw)
{
    const int lane = threadIdx.x & 31;
    const int rlo = dlo >= 1 ? (dlo - 1) / TI : 0, rhi = min(nrb - 1, dhi / TI);
    const int clo = dlo >= 1 ? (dlo - 1) / TJ : 0, chi = min(ncc - 1, dhi / TJ);
    const int nR = rhi - rlo + 1, nC = chi - clo + 1;
    for (int task = gw; task < nR + nC; task += nw) {
        if (task < nR) {
            const int rb = rlo + task;
            const Box b = warp_box_mirror(P, E, rb * TI, min(rb * TI + TI, n - 1), i, j);
            if (lane == 0) rbox[rb] = b;
        } else {
            const int cc = clo + task - nR;
            const Box b = warp_box_mirror(P, E, cc * TJ, min(cc * TJ + TJ, n), i, j);
            if (lane == 0) cbox[cc] = b;
        }
    }
}

// Group minima for the sweep whose dirty positions are [dlo, dhi] (dirty row
// blocks [rlo, rhi], chunks [clo, chi]), one warp per row block (warps gw of
// nw): a dirty row block's groups are reset to none; in a clean row block a
// group inside [clo, chi] is reset to none, a group partly inside is set to
// the min over its clean tiles (read from tb2), and both those and the
// untouched groups' sm2 enter the returned warp minimum (every lane).
__device__ __forceinline__ unsigned long long group_minima(const unsigned long long* tb2, unsigned long long* sm2,
                                                           int nrb, int ncc, int nsc, int rlo, int rhi, int clo,
                                                           int chi, int gw, int nw)
{
    const int lane = threadIdx.x & 31;
    unsigned long long m = kKeyNone;
    const int sclo = clo / kGroupChunks, schi = chi / kGroupChunks;
    for (int rb = gw; rb < nrb; rb += nw) {
        unsigned long long* srow = sm2 + (long long)rb * nsc;
        if (rb >= rlo && rb <= rhi) {
            for (int sc = lane; sc < nsc; sc += 32) srow[sc] = kKeyNone;
            continue;
        }
        // the partly dirty groups (sclo, schi): their clean tiles, two loads per lane each
        unsigned long long ga = kKeyNone, gb = kKeyNone;
        const unsigned long long* trow = tb2 + (long long)rb * ncc;
#pragma unroll
        for (int h = 0; h < kGroupChunks / 32; h++) {
            const int ca = sclo * kGroupChunks + h * 32 + lane, cb = schi * kGroupChunks + h * 32 + lane;
            const unsigned long long va = (ca < ncc && (ca < clo || ca > chi)) ? trow[ca] : kKeyNone;
            const unsigned long long vb = (cb < ncc && (cb < clo || cb > chi)) ? trow[cb] : kKeyNone;
            ga = min(ga, va);
            gb = min(gb, vb);
        }
        for (int sc = lane; sc < nsc; sc += 32) {
            if (sc == sclo || sc == schi) continue;
            if (sc > sclo && sc < schi) srow[sc] = kKeyNone;  // every tile of the group is dirty
            else m = min(m, srow[sc]);
        }
        for (int o = 16; o > 0; o >>= 1) {
            ga = min(ga, __shfl_xor_sync(0xffffffffu, ga, o));
            gb = min(gb, __shfl_xor_sync(0xffffffffu, gb, o));
        }
        if (lane == 0) {
            srow[sclo] = ga;
            if (schi != sclo) srow[schi] = gb;
        }
        m = min(m, min(ga, gb));
    }
    for (int o = 16; o > 0; o >>= 1) m = min(m, __shfl_xor_sync(0xffffffffu, m, o));
    return m;
}

constexpr int kBoxWarps = 4;  // (X): warps per CTA computing boxes; the others scan the group minima

template <int R, bool FIRST>
__global__ void __launch_bounds__(512, 1) inc_ls2_kernel(float2* P0, int* E0, int* T0, float2* P1, int* E1, int* T1,
                                                         int n, int np, const int* __restrict__ tmap, int TI, int TJ,
                                                         int nrb, int ncc, int nsc, Box* rbox, Box* cbox,
                                                         unsigned long long* tb2, unsigned long long* sm2,
                                                         unsigned long long* ctr, Slot* slots, int parity,
                                                         long long max_moves, long long budget, int full, int* ctl,
                                                         int flags, unsigned long long* trace, long long trace_cap,
                                                         int tile_bytes, int part_cols)
{
    extern __shared__ float4 smem[];
    const int wib = threadIdx.x >> 5, nwb = blockDim.x >> 5, lane = threadIdx.x & 31;
    const int gw = blockIdx.x * nwb + wib, nw = gridDim.x * nwb;
    const int gtid = blockIdx.x * blockDim.x + threadIdx.x, stride = gridDim.x * blockDim.x;
    const bool boxw = wib < kBoxWarps;  // (X) role
    const int gwb = blockIdx.x * kBoxWarps + wib, nwbx = gridDim.x * kBoxWarps;
    const int gwc = blockIdx.x * (nwb - kBoxWarps) + (wib - kBoxWarps), nwc = gridDim.x * (nwb - kBoxWarps);
    const int tflags = (flags | kSweepLocal) & ~kSweepSeed;
    __shared__ Slot s_in;
    __shared__ unsigned long long s_min[32];
    unsigned long long target = 0;
    int p = parity;
    float2 *Pc = P0, *Pa = P1;
    int *Ec = E0, *Ea = E1, *Tc = T0, *Ta = T1;
#ifdef TSP2OPT_PHASE_TIMING
    // CTA 0's cycles per phase ([0] C, [1] barrier, [2] X, [3] barrier) and the per-move
    // maxima over CTAs ([8] C, [9] X); [10] moves counted
    const bool t_lead = threadIdx.x == 0, t_cta0 = blockIdx.x == 0 && threadIdx.x == 0;
#endif
    // prologue: the first sweep's dirty set, its boxes and group minima; alternate := current
    if (threadIdx.x == 0) {
        s_in.done = *(volatile int*)&slots[p].done;
        s_in.seed_ok = full ? 0 : *(volatile int*)&slots[p].seed_ok;
        s_in.last_key = *(volatile unsigned long long*)&slots[p].last_key;
    }
    __syncthreads();
    if (s_in.done) {
        if (gtid == 0) ctl[0] = p;
        return;  // uniform
    }
    int dlo = 0, dhi = n;
    if (s_in.seed_ok) {
        dlo = key_i(s_in.last_key);
        dhi = key_j(s_in.last_key);
    }
    int rlo = dlo >= 1 ? (dlo - 1) / TI : 0, rhi = min(nrb - 1, dhi / TI);
    int clo = dlo >= 1 ? (dlo - 1) / TJ : 0, chi = min(ncc - 1, dhi / TJ);
    dirty_boxes(Pc, Ec, n, TI, TJ, nrb, ncc, dlo, dhi, -1, -1, rbox, cbox, gw, nw);
    {
        unsigned long long m = group_minima(tb2, sm2, nrb, ncc, nsc, rlo, rhi, clo, chi, gw, nw);
        if (lane == 0) s_min[wib] = s_in.seed_ok ? m : kKeyNone;
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned long long bm = s_min[0];
            for (int w = 1; w < nwb; w++) bm = min(bm, s_min[w]);
            if (!s_in.seed_ok) {
                if (blockIdx.x == 0) slots[p].key = seed_key();  // full sweep: nothing is clean
            } else if (bm != kKeyNone) {
                atomicMin(&slots[p].key, bm);
            }
        }
    }
    for (int k = gtid; k < np; k += stride) {
        Pa[k] = Pc[k];
        Ea[k] = Ec[k];
        Ta[k] = Tc[k];
    }
    grid_sync_mono(ctr, target);
    int ip = -1, jp = -1;  // the launch's previous move: where the two buffers differ
    for (long long it = 0; it < budget; it++) {
        Slot* in = slots + p;
        Slot* out = slots + (p ^ 1);
#ifdef TSP2OPT_PHASE_TIMING
        const long long tc0 = clock64();
#endif
        // (C) cull + sweep the dirty tiles of the current state into in->key
        if (gtid == 0) out->key = seed_key();  // read last by the previous (X), before the barrier
        {
            const long long nA = (long long)(rhi - rlo + 1) * ncc;
            const long long nB = (long long)nrb * (chi - clo + 1);
            inc_kept_parts<R, FIRST>(Pc, Ec, n, tmap, TI, TJ, nrb, ncc, rlo, rhi, clo, chi, nA, nB, rbox, cbox, in,
                                     nullptr, tflags, part_cols, smem, tile_bytes, tb2, sm2, nsc);
        }
#ifdef TSP2OPT_PHASE_TIMING
        const long long tc1 = clock64();
        if (t_lead) atomicMax(&g_phase_it[0], (unsigned long long)(tc1 - tc0));
        if (t_cta0) atomicAdd(&g_phase[0], (unsigned long long)(tc1 - tc0));
#endif
        grid_sync_mono(ctr, target);
#ifdef TSP2OPT_PHASE_TIMING
        const long long tx0 = clock64();
        if (t_cta0) {
            atomicAdd(&g_phase[1], (unsigned long long)(tx0 - tc1));
            g_phase[8] += g_phase_it[0];
            g_phase_it[0] = 0;
            for (int q = 2; q < 6; q++) {
                g_phase[10 + q] += g_phase_it[q];
                g_phase_it[q] = 0;
            }
        }
#endif
        // (X) decide and apply the winning move out of place; prepare the next sweep
        if (threadIdx.x == 0) {
            s_in.key = *(volatile unsigned long long*)&in->key;
            s_in.moves = *(volatile long long*)&in->moves;
            s_in.length = *(volatile long long*)&in->length;
            s_in.done = *(volatile int*)&in->done;
        }
        __syncthreads();
        const unsigned long long key = s_in.key;
        const int i = key_i(key), j = key_j(key);
        const long long moves = s_in.moves;
        const bool apply = !s_in.done && key_delta(key) < 0 && moves < max_moves;
        // the slot, the trace and the apply's few writes go to the last CTA's last threads: warps
        // without a box or group task (the others' critical path is the box / group round trips)
        const int rtid = stride - 1 - gtid;
        if (rtid == 0) {
            out->last_key = key;
            out->moves = moves;
            out->length = s_in.length;
            out->done = s_in.done;
            out->next_tile = 0;
            out->ncull = 0;
            out->mtype = 0;
            out->seed_ok = apply ? 1 : 0;
            if (!s_in.done) {
                if (key_delta(key) >= 0) out->done = 1;      // local minimum (reading R7)
                else if (moves >= max_moves) out->done = 2;  // capped with an improving move left (R8)
            }
            if (apply) {  // exact delta from the current state (a first-improvement key carries a marker)
                const int di = exact_dist_biased(Pc[i], Pc[j]), dj = exact_dist_biased(Pc[i + 1], Pc[j + 1]);
                const int d = di + dj - Ec[i] - Ec[j];
                out->length = s_in.length + d;
                out->moves = moves + 1;
                out->last_key = pack_key(d, i, j);
                if (trace && moves < trace_cap) trace[moves] = out->last_key;
            }
        }
        if (apply) {
            // P / tour: positions [i+1, j] reversed, [ip+1, jp] brought up to date
            const int n1 = j - i, n2 = ip >= 0 ? jp - ip : 0;
            for (int t = rtid; t < n1 + n2; t += stride) {
                const int k = t < n1 ? i + 1 + t : ip + 1 + (t - n1);
                const int mk = (k > i && k <= j) ? i + j + 1 - k : k;
                Pa[k] = Pc[mk];
                Ta[k] = Tc[mk];
            }
            // e: [i, j] (the two new edges, the inside reversed), [ip, jp] brought up to date
            const int m1 = j - i + 1, m2 = ip >= 0 ? jp - ip + 1 : 0;
            for (int t = rtid; t < m1 + m2; t += stride) {
                const int k = t < m1 ? i + t : ip + (t - m1);
                if (k == i) Ea[k] = exact_dist_biased(Pc[i], Pc[j]);
                else if (k == j) Ea[k] = exact_dist_biased(Pc[i + 1], Pc[j + 1]);
                else Ea[k] = (k > i && k < j) ? Ec[i + j - k] : Ec[k];
            }
            rlo = i >= 1 ? (i - 1) / TI : 0;
            rhi = min(nrb - 1, j / TI);
            clo = i >= 1 ? (i - 1) / TJ : 0;
            chi = min(ncc - 1, j / TJ);
            unsigned long long m = kKeyNone;
            if (boxw) dirty_boxes(Pc, Ec, n, TI, TJ, nrb, ncc, i, j, i, j, rbox, cbox, gwb, nwbx);
            else m = group_minima(tb2, sm2, nrb, ncc, nsc, rlo, rhi, clo, chi, gwc, nwc);
            if (lane == 0) s_min[wib] = m;
            __syncthreads();
            if (threadIdx.x == 0) {
                unsigned long long bm = s_min[0];
                for (int w = 1; w < nwb; w++) bm = min(bm, s_min[w]);
                if (bm != kKeyNone) atomicMin(&out->key, bm);
            }
        }
#ifdef TSP2OPT_PHASE_TIMING
        const long long tx1 = clock64();
        if (t_lead) atomicMax(&g_phase_it[1], (unsigned long long)(tx1 - tx0));
        if (t_cta0) atomicAdd(&g_phase[2], (unsigned long long)(tx1 - tx0));
#endif
        p ^= 1;
        grid_sync_mono(ctr, target);
#ifdef TSP2OPT_PHASE_TIMING
        if (t_cta0) {
            atomicAdd(&g_phase[3], (unsigned long long)(clock64() - tx1));
            g_phase[9] += g_phase_it[1];
            g_phase_it[1] = 0;
            g_phase[10] += 1;
        }
#endif
        if (!apply) break;  // uniform: every CTA read the same key
        ip = i;
        jp = j;
        float2* tp = Pc;
        Pc = Pa;
        Pa = tp;
        int* te = Ec;
        Ec = Ea;
        Ea = te;
        int* tt = Tc;
        Tc = Ta;
        Ta = tt;
    }
    // the handle's buffers: copy the last move's positions back if the current state is the alternate
    if (Pc != P0 && ip >= 0) {
        for (int t = gtid; t < jp - ip; t += stride) {
            P0[ip + 1 + t] = Pc[ip + 1 + t];
            T0[ip + 1 + t] = Tc[ip + 1 + t];
        }
        for (int t = gtid; t <= jp - ip; t += stride) E0[ip + t] = Ec[ip + t];
    }
    if (gtid == 0) ctl[0] = p;
}

// ===========================================================================
// Persistent incremental local search, ONE grid barrier per move
// (inc_ls1_kernel).  Phase m decides move m from the key the previous phase
// completed, then, all reading only the pre-move state S_{m-1}:
//   * item warps (14 per CTA) cull the tiles move m dirties, stage the kept
//     ones through the reversal's mirror map (new P[k] = P[i+j+1-k] on
//     [i+1, j], new e[k] = e[i+j-k] on (i, j), the two new edges) and sweep
//     them in column parts: the minima of S_m, written to the dense tile
//     minima and the next key.  The cull uses CONSERVATIVE boxes for the
//     dirty blocks: the union of the stored boxes of the blocks its new
//     cities and edges come from (and of the block itself unless the move
//     replaces all of it), and the largest of their edges and the two new
//     ones -- a superset of what S_m's exact boxes keep, so every tile that
//     can hold an improving pair is swept;
//   * side warps (2 per CTA) write S_m into the other P / E / tour buffer (the
//     positions of moves m-1 and m), compute S_m's exact boxes of the dirty
//     blocks into the other box buffer (copying the blocks move m-1 dirtied),
//     and fold the clean tiles' minima into the next key through the group
//     minima (a group touched by move m is marked invalid; an invalid group
//     that move m leaves clean is recomputed from its tiles first).
// The key is triple-buffered (read, written, reset in the same phase), so one
// barrier per move orders everything; the result is the same move sequence as
// the two- and three-barrier kernels.  A launch starts with a full sweep of its
// state and leaves seed_ok = 0 (the next launch starts full).
// ===========================================================================
#ifndef TSP2OPT_SIDE_WARPS
#define TSP2OPT_SIDE_WARPS 2  // measured: 2 of 16 warps for the apply, boxes and group minima beat 4 and 1
#endif
constexpr int kSideWarps = TSP2OPT_SIDE_WARPS;  // inc_ls1: per CTA, the rest sweep
constexpr unsigned long long kGroupInvalid = 0;  // not a key (delta + 2^18 > 0): "recompute this group"

// Conservative box of block `b` (positions [b*B, min(b*B + B, last)], edges up
// to the block end - 1) of the state after move (i, j), from the stored boxes
// of the state before it: the union with the blocks whose positions the
// reversal maps into this block, and the two new edges.
__device__ __forceinline__ Box cons_box(const Box* boxes, int b, int B, int nb, int last, int i, int j, int di,
                                        int dj)
{
    if (i < 0) return boxes[b];
    const int a0 = b * B, a1 = min(a0 + B, last);
    Box r;
    if (a0 >= i + 1 && a1 <= j) {  // every city and edge of the block is replaced: the sources only
        r.xlo = r.ylo = 1 << 30;
        r.xhi = r.yhi = -1;
        r.emax = 0;
    } else {
        r = boxes[b];
    }
    const int lo = max(a0, i + 1), hi = min(a1, j);
    if (lo <= hi) {  // positions [lo, hi] receive cities from [i+j+1-hi, i+j+1-lo], edges from one lower
        const int s0 = max(0, (i + j - hi) / B), s1 = min(nb - 1, (i + j + 1 - lo) / B);
        for (int s = s0; s <= s1; s++) {
            const Box q = boxes[s];
            r.xlo = min(r.xlo, q.xlo);
            r.xhi = max(r.xhi, q.xhi);
            r.ylo = min(r.ylo, q.ylo);
            r.yhi = max(r.yhi, q.yhi);
            r.emax = max(r.emax, q.emax);
        }
    }
    if (i >= a0 && i < a1) r.emax = max(r.emax, di);
    if (j >= a0 && j < a1) r.emax = max(r.emax, dj);
    return r;
}

template <int NT>
__device__ __forceinline__ void bar_items()
{
    asm volatile("bar.sync 1, %0;" ::"n"(NT) : "memory");
}

// The item warps' share of phase m: cull / stage / sweep the tiles move (i, j)
// dirties (i < 0: every tile, plain reads), into tb2 and *key.
template <int R, bool FIRST, int NT>
__device__ __forceinline__ void inc1_items(const float2* P, const int* E, int n, const int* __restrict__ tmap, int TI,
                                           int TJ, int nrb, int ncc, int i, int j, int di, int dj, const Box* rbox,
                                           const Box* cbox, unsigned long long* key, unsigned long long* tb2,
                                           int tflags, int part_cols, float4* smem, int tile_bytes)
{
    __shared__ int s_nk;
    __shared__ int4 s_kt[NT];
    __shared__ unsigned long long s_tmin[kStageTiles];
    const int tid = threadIdx.x, wib = tid >> 5, nwi = NT / 32;
    const int dlo = i < 0 ? 0 : i, dhi = i < 0 ? n : j;
    const int rlo = dlo >= 1 ? (dlo - 1) / TI : 0, rhi = min(nrb - 1, dhi / TI);
    const int clo = dlo >= 1 ? (dlo - 1) / TJ : 0, chi = min(ncc - 1, dhi / TJ);
    const long long nA = (long long)(rhi - rlo + 1) * ncc, nB = (long long)nrb * (chi - clo + 1);
    const int nparts = (TJ + part_cols - 1) / part_cols;
    const long long step = (long long)NT * gridDim.x;
    for (long long base = 0; base < nA + nB; base += step) {
        if (tid == 0) s_nk = 0;
        bar_items<NT>();
        const long long u = base + (long long)tid * gridDim.x + blockIdx.x;
        if (u < nA + nB) {
            int rb, cc;
            bool cand = true;
            if (u < nA) {
                rb = rlo + (int)(u / ncc);
                cc = (int)(u % ncc);
            } else {
                const long long v = u - nA;
                rb = (int)(v / (chi - clo + 1));
                cc = clo + (int)(v % (chi - clo + 1));
                cand = rb < rlo || rb > rhi;
            }
            if (cand) {
                const int t = tmap[(long long)rb * ncc + cc];
                const Box r = (rb >= rlo && rb <= rhi) ? cons_box(rbox, rb, TI, nrb, n - 1, i, j, di, dj) : rbox[rb];
                const Box c = (cc >= clo && cc <= chi) ? cons_box(cbox, cc, TJ, ncc, n, i, j, di, dj) : cbox[cc];
                if (t >= 0) {
                    const long long gx = max(0, max(c.xlo - r.xhi, r.xlo - c.xhi));
                    const long long gy = max(0, max(c.ylo - r.yhi, r.ylo - c.yhi));
                    const long long T = (long long)max(r.emax, c.emax) - 1;
                    if (T >= 0 && gx * gx + gy * gy <= T * T + T) s_kt[atomicAdd(&s_nk, 1)] = make_int4(t, rb, cc, 0);
                    else tb2[(long long)rb * ncc + cc] = kKeyNone;
                }
            }
        }
        bar_items<NT>();
        const int nk = s_nk;
        for (int b0 = 0; b0 < nk; b0 += kStageTiles) {
            const int nb = min(kStageTiles, nk - b0);
            const int ncolp = TJ + 2, nrowp = 32 * R + 1, per = ncolp + nrowp;
            constexpr int U = 8;
            for (int x0 = 0; x0 < nb * per; x0 += U * NT) {
                float2 pv[U];
                int ev[U];
#pragma unroll
                for (int v = 0; v < U; v++) {
                    const int x = x0 + v * NT + tid;
                    pv[v] = make_float2(0.f, 0.f);
                    ev[v] = 0;
                    if (x < nb * per) {
                        const int k = x / per, q = x - k * per;
                        const int4 kt = s_kt[b0 + k];
                        const int pos = q < ncolp ? kt.z * TJ + q : kt.y * TI + (q - ncolp);
                        // the state after the move, read through the mirror map
                        const int mp = (pos > i && pos <= j) ? i + j + 1 - pos : pos;
                        pv[v] = P[mp];
                        ev[v] = (pos == i) ? di : (pos == j) ? dj : E[(pos > i && pos < j) ? i + j - pos : pos];
                    }
                }
#pragma unroll
                for (int v = 0; v < U; v++) {
                    const int x = x0 + v * NT + tid;
                    if (x < nb * per) {
                        const int k = x / per, q = x - k * per;
                        const TileSmem tsm(reinterpret_cast<char*>(smem) + (size_t)k * tile_bytes, TJ, 32 * R);
                        if (q < ncolp) {
                            tsm.put(q, pv[v], (float)ev[v]);
                        } else {
                            const int rq = q - ncolp;
                            const int ln = rq / R, sl = rq - ln * R;
                            if (ln < 32) {
                                tsm.rowp[ln * (R + 1) + sl] = pv[v];
                                tsm.rowe[rq] = (float)ev[v];
                            }
                            if (sl == 0 && ln > 0) tsm.rowp[(ln - 1) * (R + 1) + R] = pv[v];
                        }
                    }
                }
            }
            if (tid < nb) s_tmin[tid] = kKeyNone;
            bar_items<NT>();
            for (int it = wib; it < nb * nparts; it += nwi) {
                const int k = it / nparts, part = it - k * nparts;
                const int4 kt = s_kt[b0 + k];
                const TileSmem tsm(reinterpret_cast<char*>(smem) + (size_t)k * tile_bytes, TJ, 32 * R);
                const int I0 = kt.y * TI, J0 = kt.z * TJ, J1 = min(J0 + TJ, n);
                const int jb = J0 + part * part_cols, je = min(jb + part_cols, J1);
                if (jb < je) {
                    const unsigned long long mk = sweep_part<R, FIRST>(I0, J0, jb, je, tsm, tflags);
                    if (mk != kKeyNone) atomicMin(&s_tmin[k], mk);
                }
            }
            bar_items<NT>();
            if (tid < nb) {
                const unsigned long long m = s_tmin[tid];
                const int4 kt = s_kt[b0 + tid];
                tb2[(long long)kt.y * ncc + kt.z] = m;
                if (m != kKeyNone) atomicMin(key, m);
            }
            bar_items<NT>();
        }
    }
}

// The side warps' group minima for the sweep after move (i, j) (i < 0: none --
// everything is dirty and was invalidated): one lane per group, the groups
// that need their tiles read (invalid ones move m leaves clean: recomputed and
// stored; partly dirty ones: their clean tiles) collected per warp and read by
// the whole warp.  Returns the warp's minimum over the clean tiles (all lanes).
__device__ __forceinline__ unsigned long long inc1_groups(unsigned long long* tb2, unsigned long long* sm2, int nrb,
                                                          int ncc, int nsc, int TI, int TJ, int n, int i, int j,
                                                          int gw, int nw)
{
    const int lane = threadIdx.x & 31;
    const int rlo = i >= 1 ? (i - 1) / TI : 0, rhi = min(nrb - 1, j / TI);
    const int clo = i >= 1 ? (i - 1) / TJ : 0, chi = min(ncc - 1, j / TJ);
    const long long G = (long long)nrb * nsc;
    unsigned long long m = kKeyNone;
    // group g = gw + nw * (k0 + lane): consecutive groups (a whole invalid row block) on different warps
    for (long long k0 = 0; gw + (long long)nw * k0 < G; k0 += 32) {
        const long long g = gw + (long long)nw * (k0 + lane);
        bool heavy = false, store = false;
        if (g < G) {
            const int rb = (int)(g / nsc), sc = (int)(g % nsc);
            const int c0 = sc * kGroupChunks, c1 = min(c0 + kGroupChunks, ncc) - 1;
            if (rb >= rlo && rb <= rhi) {
                sm2[g] = kGroupInvalid;
            } else if (c0 <= chi && c1 >= clo) {
                if (c0 >= clo && c1 <= chi) sm2[g] = kGroupInvalid;
                else {
                    heavy = true;  // partly dirty: its clean tiles; stays invalid
                    sm2[g] = kGroupInvalid;
                }
            } else {
                const unsigned long long v = sm2[g];
                if (v == kGroupInvalid) heavy = store = true;
                else m = min(m, v);
            }
        }
        unsigned hv = __ballot_sync(0xffffffffu, heavy);
        const unsigned sv = __ballot_sync(0xffffffffu, store);
        while (hv) {
            const int src = __ffs(hv) - 1;
            hv &= hv - 1;
            const long long gg = gw + (long long)nw * (k0 + src);
            const int rb = (int)(gg / nsc), sc = (int)(gg % nsc);
            const unsigned long long* trow = tb2 + (long long)rb * ncc;
            unsigned long long gm = kKeyNone;
#pragma unroll
            for (int h = 0; h < kGroupChunks / 32; h++) {
                const int cc = sc * kGroupChunks + h * 32 + lane;
                if (cc < ncc && (cc < clo || cc > chi)) gm = min(gm, trow[cc]);
            }
            for (int o = 16; o > 0; o >>= 1) gm = min(gm, __shfl_xor_sync(0xffffffffu, gm, o));
            if (lane == src && ((sv >> src) & 1u)) sm2[gg] = gm;  // recomputed (all its tiles are clean)
            m = min(m, gm);
        }
    }
    for (int o = 16; o > 0; o >>= 1) m = min(m, __shfl_xor_sync(0xffffffffu, m, o));
    return m;
}

template <int R, bool FIRST>
__global__ void __launch_bounds__(512, 1) inc_ls1_kernel(float2* P0, int* E0, int* T0, float2* P1, int* E1, int* T1,
                                                         int n, int np, const int* __restrict__ tmap, int TI, int TJ,
                                                         int nrb, int ncc, int nsc, Box* rboxA, Box* cboxA,
                                                         Box* rboxB, Box* cboxB, unsigned long long* tb2,
                                                         unsigned long long* sm2, unsigned long long* ctr,
                                                         unsigned long long* keys3, Slot* slots, int parity,
                                                         long long max_moves, long long budget, int* ctl, int flags,
                                                         unsigned long long* trace, long long trace_cap,
                                                         int tile_bytes, int part_cols)
{
    extern __shared__ float4 smem[];
    constexpr int NT = 32 * (16 - kSideWarps);  // item threads per CTA
    const int wib = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int gtid = blockIdx.x * blockDim.x + threadIdx.x, stride = gridDim.x * blockDim.x;
    const bool side = wib >= 16 - kSideWarps;
    const int gws = blockIdx.x * kSideWarps + (wib - (16 - kSideWarps)), nws = gridDim.x * kSideWarps;
    const int gw = blockIdx.x * 16 + wib, nw = gridDim.x * 16;
    const int tflags = (flags | kSweepLocal) & ~kSweepSeed;
    __shared__ Slot s_in;
    __shared__ int s_d[2];
    unsigned long long target = 0;
    float2 *Pc = P0, *Pa = P1;
    int *Ec = E0, *Ea = E1, *Tc = T0, *Ta = T1;
    Box *rbc = rboxA, *cbc = cboxA, *rba = rboxB, *cba = cboxB;
    if (threadIdx.x == 0) {
        s_in.done = *(volatile int*)&slots[parity].done;
        s_in.moves = *(volatile long long*)&slots[parity].moves;
        s_in.length = *(volatile long long*)&slots[parity].length;
    }
    __syncthreads();
    if (s_in.done) {
        if (gtid == 0) ctl[0] = parity;
        return;  // uniform
    }
    long long moves = s_in.moves, length = s_in.length;
    int done = 0;
    unsigned long long klast = seed_key();
    // prologue: every block's box (both buffers), alternate := current, all groups invalid
    {
        for (int task = gw; task < nrb + ncc; task += nw) {
            if (task < nrb) {
                const Box b = warp_box_mirror(Pc, Ec, task * TI, min(task * TI + TI, n - 1), -1, -1);
                if (lane == 0) rbc[task] = rba[task] = b;
            } else {
                const int cc = task - nrb;
                const Box b = warp_box_mirror(Pc, Ec, cc * TJ, min(cc * TJ + TJ, n), -1, -1);
                if (lane == 0) cbc[cc] = cba[cc] = b;
            }
        }
        for (long long g = gtid; g < (long long)nrb * nsc; g += stride) sm2[g] = kGroupInvalid;
        for (int k = gtid; k < np; k += stride) {
            Pa[k] = Pc[k];
            Ea[k] = Ec[k];
            Ta[k] = Tc[k];
        }
        if (gtid == 0) keys3[1] = seed_key();
    }
    grid_sync_mono(ctr, target);
    int ip = -1, jp = -1;  // the previous move: where the two P / E / tour buffers differ
    int kr = 0, kw = 1, kz = 2;
    for (long long it = 0; it <= budget; it++) {
        int i = -1, j = -1, di = 0, dj = 0;
        bool apply = false;
        if (it > 0) {  // decide move m from the completed key
            if (threadIdx.x == 0) {
                s_in.key = *(volatile unsigned long long*)&keys3[kr];
                const int ki = key_i(s_in.key), kj = key_j(s_in.key);
                s_d[0] = exact_dist_biased(Pc[ki], Pc[kj]);
                s_d[1] = exact_dist_biased(Pc[ki + 1], Pc[kj + 1]);
            }
            __syncthreads();
            const unsigned long long key = s_in.key;
            klast = key;
            if (key_delta(key) >= 0) done = 1;         // local minimum (reading R7)
            else if (moves >= max_moves) done = 2;     // capped with an improving move left (R8)
            else if (it == budget) done = 0;           // launch budget: the next launch resumes (full)
            else apply = true;
            if (!apply) break;  // uniform
            i = key_i(key);
            j = key_j(key);
            di = s_d[0];
            dj = s_d[1];
            if (gtid == 0) {  // the exact delta (a first-improvement key carries a marker): thread 0 only
                const int d = di + dj - Ec[i] - Ec[j];
                klast = pack_key(d, i, j);
                if (trace && moves < trace_cap) trace[moves] = klast;
                length += d;
            }
            moves += 1;
        }
        if (gtid == 0) keys3[kz] = seed_key();  // read in the previous phase, written in the next
        if (!side) {
            inc1_items<R, FIRST, NT>(Pc, Ec, n, tmap, TI, TJ, nrb, ncc, i, j, di, dj, rbc, cbc, &keys3[kw], tb2,
                                     tflags, part_cols, smem, tile_bytes);
        } else if (apply) {
            // (1) S_m into the alternate buffers: positions of moves m-1 and m
            const int sid = gws * 32 + lane, sn = nws * 32;
            const int n1 = j - i, n2 = ip >= 0 ? jp - ip : 0;
            for (int t = sid; t < n1 + n2; t += sn) {
                const int k = t < n1 ? i + 1 + t : ip + 1 + (t - n1);
                const int mk = (k > i && k <= j) ? i + j + 1 - k : k;
                Pa[k] = Pc[mk];
                Ta[k] = Tc[mk];
            }
            const int m1 = j - i + 1, m2 = ip >= 0 ? jp - ip + 1 : 0;
            for (int t = sid; t < m1 + m2; t += sn) {
                const int k = t < m1 ? i + t : ip + (t - m1);
                Ea[k] = k == i ? di : k == j ? dj : (k > i && k < j) ? Ec[i + j - k] : Ec[k];
            }
            // (2) S_m's exact boxes of the blocks move m dirties; move m-1's blocks copied over
            {
                const int rlo = i >= 1 ? (i - 1) / TI : 0, rhi = min(nrb - 1, j / TI);
                const int clo = i >= 1 ? (i - 1) / TJ : 0, chi = min(ncc - 1, j / TJ);
                const int nR = rhi - rlo + 1, nC = chi - clo + 1;
                for (int task = gws; task < nR + nC; task += nws) {
                    if (task < nR) {
                        const int rb = rlo + task;
                        const Box b = warp_box_mirror(Pc, Ec, rb * TI, min(rb * TI + TI, n - 1), i, j);
                        if (lane == 0) rba[rb] = b;
                    } else {
                        const int cc = clo + task - nR;
                        const Box b = warp_box_mirror(Pc, Ec, cc * TJ, min(cc * TJ + TJ, n), i, j);
                        if (lane == 0) cba[cc] = b;
                    }
                }
                if (ip >= 0) {
                    const int qlo = ip >= 1 ? (ip - 1) / TI : 0, qhi = min(nrb - 1, jp / TI);
                    const int plo = ip >= 1 ? (ip - 1) / TJ : 0, phi = min(ncc - 1, jp / TJ);
                    const int sid2 = gws * 32 + lane;
                    for (int t = sid2; t < (qhi - qlo + 1) + (phi - plo + 1); t += sn) {
                        if (t <= qhi - qlo) {
                            const int rb = qlo + t;
                            if (rb < rlo || rb > rhi) rba[rb] = rbc[rb];
                        } else {
                            const int cc = plo + t - (qhi - qlo + 1);
                            if (cc < clo || cc > chi) cba[cc] = cbc[cc];
                        }
                    }
                }
            }
            // (3) the clean tiles' minima of S_m
            const unsigned long long m = inc1_groups(tb2, sm2, nrb, ncc, nsc, TI, TJ, n, i, j, gws, nws);
            if (lane == 0 && m != kKeyNone) atomicMin(&keys3[kw], m);
        }
        grid_sync_mono(ctr, target);
        kr = (kr + 1) % 3;
        kw = (kw + 1) % 3;
        kz = (kz + 1) % 3;
        if (apply) {
            ip = i;
            jp = j;
            float2* tp = Pc;
            Pc = Pa;
            Pa = tp;
            int* te = Ec;
            Ec = Ea;
            Ea = te;
            int* tt = Tc;
            Tc = Ta;
            Ta = tt;
            Box* tb = rbc;
            rbc = rba;
            rba = tb;
            tb = cbc;
            cbc = cba;
            cba = tb;
        }
    }
    // the handle's buffers: copy the last move's positions back if the current state is the alternate
    if (Pc != P0 && ip >= 0) {
        for (int t = gtid; t < jp - ip; t += stride) {
            P0[ip + 1 + t] = Pc[ip + 1 + t];
            T0[ip + 1 + t] = Tc[ip + 1 + t];
        }
        for (int t = gtid; t <= jp - ip; t += stride) E0[ip + t] = Ec[ip + t];
    }
    if (gtid == 0) {
        Slot o;
        o.key = seed_key();
        o.last_key = klast;
        o.moves = moves;
        o.length = length;
        o.done = done;
        o.next_tile = 0;
        o.ncull = 0;
        o.seed_ok = 0;  // the next launch starts with a full sweep
        o.mtype = 0;
        slots[parity] = o;
        ctl[0] = parity;
    }
}

// ===========================================================================
// Persistent dense local search with dynamic tile claims (medium n, one GPU):
// one cooperative launch of one 16-warp CTA per SM; per iteration every WARP
// claims tiles of the dense tiling from the slot's counter (largest first) and
// sweeps each with its private shared memory and the in-sweep bound (the slot's
// running key), then one grid barrier, the apply, another barrier.  The round-
// robin tile assignment of local_search_kernel lost to the per-iteration
// kernels from n ~ 7e3 because static shares of unequal tiles imbalance; the
// claims balance them, and two barriers replace two launches per move.
// ===========================================================================
template <int R>
__global__ void __launch_bounds__(512, 1) dense_ls_kernel(float2* __restrict__ P, int* __restrict__ E,
                                                          int* __restrict__ tour, int n,
                                                          const int2* __restrict__ tiles, int ntiles, int TJ,
                                                          Slot* __restrict__ slots, int parity, long long max_moves,
                                                          long long budget, unsigned* __restrict__ bar,
                                                          int* __restrict__ ctl, int flags,
                                                          unsigned long long* __restrict__ tilebest,
                                                          unsigned long long* __restrict__ trace, long long trace_cap,
                                                          int tile_bytes)
{
    extern __shared__ float4 smem[];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const TileSmem sm(reinterpret_cast<char*>(smem) + (size_t)wib * tile_bytes, TJ, 32 * R);
    const int gtid = blockIdx.x * blockDim.x + threadIdx.x, stride = gridDim.x * blockDim.x;
    const int tflags = flags & ~(kSweepSeed | kSweepLocal | kSweepIncremental);
    __shared__ Slot s_in;
    int p = parity;
    for (long long it = 0; it < budget; it++) {
        Slot* in = slots + p;
        if (threadIdx.x == 0) s_in.done = *(volatile int*)&in->done;
        __syncthreads();
        if (s_in.done) break;  // uniform across the grid
#ifndef TSP2OPT_DENSE_CLAIM
#define TSP2OPT_DENSE_CLAIM 0  // tiles per claim (0: static round-robin by warp; measured best of 0 / 1 / 4 / 16)
#endif
        if (TSP2OPT_DENSE_CLAIM == 0) {
            const int gw = blockIdx.x * (blockDim.x >> 5) + wib, nw = gridDim.x * (blockDim.x >> 5);
            for (int t = gw; t < ntiles; t += nw)
                sweep_tile<R, true, false, true>(P, E, n, tiles[t], TJ, in, sm, tilebest + t, tflags);
        } else {
            // the first chunk by warp index, then claims of TSP2OPT_DENSE_CLAIM consecutive
            // (similar-sized) tiles: few atomics on the slot's counter per sweep
            const int gw = blockIdx.x * (blockDim.x >> 5) + wib, nw = gridDim.x * (blockDim.x >> 5);
            constexpr int C = TSP2OPT_DENSE_CLAIM > 0 ? TSP2OPT_DENSE_CLAIM : 1;
            int t0 = gw * C;
            for (;;) {
                if (t0 >= ntiles) break;
                for (int t = t0; t < min(t0 + C, ntiles); t++)
                    sweep_tile<R, true, false, true>(P, E, n, tiles[t], TJ, in, sm, tilebest + t, tflags);
                int c = 0;
                if (lane == 0) c = (int)atomicAdd(&in->next_tile, 1u);
                t0 = (nw + __shfl_sync(0xffffffffu, c, 0)) * C;
            }
        }
        grid_sync(bar, gridDim.x);
        if (threadIdx.x == 0) {
            s_in.key = *(volatile unsigned long long*)&in->key;
            s_in.last_key = in->last_key;
            s_in.moves = *(volatile long long*)&in->moves;
            s_in.length = *(volatile long long*)&in->length;
            s_in.done = *(volatile int*)&in->done;
            s_in.seed_ok = *(volatile int*)&in->seed_ok;
        }
        __syncthreads();
        apply_phase(P, E, tour, &s_in, slots + (p ^ 1), max_moves, 0, 0, 0, gtid, stride, trace, trace_cap, nullptr);
        p ^= 1;
        grid_sync(bar, gridDim.x);
    }
    if (gtid == 0) ctl[0] = p;
}

// ===========================================================================
// Exhaustive self-test kernels (tsp2opt_selftest).
// ===========================================================================
__global__ void selftest_dist_kernel(long long smax, unsigned long long* bad, unsigned long long* first)
{
    unsigned long long nbad = 0;
    for (long long s = (long long)blockIdx.x * blockDim.x + threadIdx.x; s <= smax;
         s += (long long)gridDim.x * blockDim.x) {
        const long long m = nint_sqrt_exact((int)s);
        if (!(m * m - m < s && s <= m * m + m) && !(s == 0 && m == 0)) {
            nbad++;
            atomicMin(first, (unsigned long long)s);
        }
    }
    if (nbad) atomicAdd(bad, nbad);
}

// Max relative error of sqrt_approx (MUFU.SQRT) over every float in [1, 2^31]
// (the float squared distances the sqrt-sum filter takes; 0 maps to 0) and a
// check that sqrt_approx(0) == 0.  Result: float bits of the max, in *out.
__global__ void selftest_sqrt_kernel(unsigned* out, unsigned* zero_bad)
{
    const unsigned lo = 0x3F800000u, hi = 0x4F000000u;  // 1.0f .. 2^31
    float worst = 0.f;
    for (unsigned u = lo + blockIdx.x * blockDim.x + threadIdx.x; u <= hi; u += gridDim.x * blockDim.x) {
        const float x = __uint_as_float(u);
        const double ex = sqrt((double)x);
        const float rel = (float)(fabs((double)sqrt_approx(x) - ex) / ex);
        worst = fmaxf(worst, rel);
    }
    atomicMax(out, __float_as_uint(worst));
    if (blockIdx.x == 0 && threadIdx.x == 0 && sqrt_approx(0.f) != 0.f) *zero_bad = 1;
}

__global__ void selftest_filter_kernel(unsigned long long* bad, unsigned long long* first)
{
    // every (dx, dy) in [0, 32767]^2; the float s is computed exactly as the
    // sweep does it (biased coordinates, FADD2 / FMUL2 / FFMA2)
    unsigned long long nbad = 0;
    const long long total = 32768LL * 32768LL;
    for (long long id = (long long)blockIdx.x * blockDim.x + threadIdx.x; id < total;
         id += (long long)gridDim.x * blockDim.x) {
        const int dx = (int)(id >> 15), dy = (int)(id & 32767);
        // row city at (dx, dy), column city at the origin; and the mirrored case
        const float2 xr = make_float2(bias_coord(dx), bias_coord(0));
        const float2 yr = make_float2(bias_coord(dy), bias_coord(0));
        const float2 ncx = make_float2(-bias_coord(0), -bias_coord(dx));
        const float2 ncy = make_float2(-bias_coord(0), -bias_coord(dy));
        const float2 s = sq2(xr, yr, ncx, ncy);
        const int t = nint_sqrt_exact(dx * dx + dy * dy);  // smallest t with "D <= t"
        const float S = sq_threshold((float)t);
        // the float nint shortcut of the rare path: when it claims a value, it is exact
        float m = -1.f;
        const float fdx = (float)dx, fdy = (float)dy;
        const bool claimed = nint_from_float(fmaf(fdx, fdx, fdy * fdy), m);
        if (!(s.x <= S) || !(s.y <= S) || (claimed && m != (float)t)) {
            nbad++;
            atomicMin(first, (unsigned long long)id);
        }
    }
    if (nbad) atomicAdd(bad, nbad);
}

// ===========================================================================
// Host-side launchers
// ===========================================================================
static std::atomic<long long> g_launches{0};

bool pdl_enabled()
{
    static const bool on = [] {
        const char* e = getenv("TSP2OPT_PDL");
        return !(e && atoi(e) == 0);
    }();
    return on;
}
template <typename... KArgs, typename... Args>
static cudaError_t launch_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                             Args... args)
{
    return launch_kernel_pdl(kernel, grid, block, smem, st, args...);
}
long long launch_count() { return g_launches.load(); }
void count_launch(int k) { g_launches += k; }

cudaError_t launch_load_tour(const int* coords, const int* tour_src, int* tour_dst, float2* P, int* E, int n,
                             Slot* slot, unsigned* stamp, unsigned epoch, cudaStream_t st)
{
    init_slot_kernel<<<1, 1, 0, st>>>(slot, 1);
    load_tour_kernel<<<(n + 255) / 256, 256, 0, st>>>(coords, tour_src, tour_dst, P, E, n, slot, stamp, epoch);
    g_launches += 2;
    return cudaGetLastError();
}

cudaError_t launch_double_bridge(const int* in, int* out, int n, int a, int b, int c, cudaStream_t st)
{
    double_bridge_kernel<<<(n + 255) / 256, 256, 0, st>>>(in, out, n, a, b, c);
    g_launches += 1;
    return cudaGetLastError();
}

// First improvement (reading R20): the sweep's min carries the marker delta
// kFirstDelta; replace it by the exact delta of the winning pair before the
// apply (length bookkeeping, trace) and the host read it.
__global__ void first_fix_kernel(const float2* __restrict__ P, const int* __restrict__ E, Slot* __restrict__ slot,
                                 int respect_done)
{
    pdl_trigger();
    pdl_wait();
    if (respect_done && *(volatile int*)&slot->done) return;
    const unsigned long long k = slot->key;
    if (key_delta(k) >= 0) return;  // the seed: no improving pair
    const int i = key_i(k), j = key_j(k);
    const int d = exact_dist_biased(P[i], P[j]) + exact_dist_biased(P[i + 1], P[j + 1]) - E[i] - E[j];
    slot->key = pack_key(d, i, j);
}

cudaError_t launch_first_fix(const float2* P, const int* E, Slot* slot, int respect_done, cudaStream_t st)
{
    cudaError_t e = launch_pdl(first_fix_kernel, dim3(1), dim3(32), 0, st, P, E, slot, respect_done);
    g_launches += 1;
    return e != cudaSuccess ? e : cudaGetLastError();
}

// Global seed of the dense sweep (tiling 0): after a move (i, j) is applied,
// every tile minimum of the sweep that found it whose pair the reversal leaves
// intact (surviving_key) is a real pair of the new tour with its exact delta.
// Their min starts the next sweep's bound for every tile at once, instead of
// the seed (0, 1, 0) that only tightens as tiles finish.  The sweep still
// examines every pair: any pair with a lower (delta, cell) replaces it.
// reeval (P, E given): every tile minimum's POSITIONS (a, b) are re-evaluated
// on the new tour instead -- (a, b) is a pair of the new tour whatever the
// move did to it, and its exact delta there (the oracle's nint arithmetic) is
// as valid a bound, from every tile instead of the surviving ones.
__global__ void __launch_bounds__(256) global_seed_kernel(const unsigned long long* __restrict__ tilebest, int ntiles,
                                                          Slot* __restrict__ slot, const float2* P, const int* E)
{
    pdl_trigger();
    pdl_wait();
    const int ok = *(volatile int*)&slot->seed_ok;
    const int done = *(volatile int*)&slot->done;
    const unsigned long long mv = *(volatile unsigned long long*)&slot->last_key;
    if (!ok || done) return;
    const int i = key_i(mv), j = key_j(mv);
    unsigned long long m = kKeyNone;
    for (int t = blockIdx.x * blockDim.x + threadIdx.x; t < ntiles; t += gridDim.x * blockDim.x) {
        const unsigned long long k = tilebest[t];
        if (!P) {
            m = min(m, surviving_key(k, i, j));
        } else if (k != kKeyNone) {
            const int a = key_i(k), b = key_j(k);
            const int d = exact_dist_biased(P[a], P[b]) + exact_dist_biased(P[a + 1], P[b + 1]) - E[a] - E[b];
            if (d < 0) m = min(m, pack_key(d, a, b));
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) m = min(m, __shfl_xor_sync(0xffffffffu, m, o));
    __shared__ unsigned long long s_m[8];
    if ((threadIdx.x & 31) == 0) s_m[threadIdx.x >> 5] = m;
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 1; w < (int)(blockDim.x >> 5); w++) m = min(m, s_m[w]);
        if (m != kKeyNone) atomicMin(&slot->key, m);
    }
}

cudaError_t launch_global_seed(const unsigned long long* tilebest, int ntiles, Slot* slot, const float2* P,
                               const int* E, cudaStream_t st)
{
    if (ntiles <= 0) return cudaSuccess;
    const int grid = std::max(1, std::min(148, (ntiles + 255) / 256));
    cudaError_t e = launch_pdl(global_seed_kernel, dim3(grid), dim3(256), 0, st, tilebest, ntiles, slot, P, E);
    g_launches += 1;
    return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_reset_key(Slot* slot, cudaStream_t st)
{
    reset_key_kernel<<<1, 1, 0, st>>>(slot);
    g_launches += 1;
    return cudaGetLastError();
}

size_t sweep_smem_bytes(const Geometry& g) { return tile_smem_bytes(g.tj, g.ti()); }
size_t sweep_smem_bytes_ps(const Geometry& g) { return tile_smem_bytes(g.tj, g.ti(), true); }

// The sweep is instantiated for R = 15 (large n: longest column steps) and
// R = 7 (small / medium n: twice the warps per row block, lower latency per
// tile); Geometry::rows selects one (choose_geometry in tsp2opt_api.cu).
static_assert(kRowsLarge == 15 && kRowsSmall == 7, "instantiated row counts");
template <typename F>
static auto by_rows(int rows, F&& f)
{
    return rows == kRowsSmall ? f(std::integral_constant<int, kRowsSmall>{})
                              : f(std::integral_constant<int, kRowsLarge>{});
}

// (R, first improvement) instantiations of the sweep kernels
template <typename F>
static auto by_rows_first(int rows, bool first, F&& f)
{
    return by_rows(rows, [&](auto r) {
        return first ? f(r, std::true_type{}) : f(r, std::false_type{});
    });
}

cudaError_t sweep_prepare()
{
    for (int R : {kRowsSmall, kRowsLarge}) {
        const Geometry gmax{R, kMaxWarps, kMaxTJ};
        for (bool first : {false, true}) {
            cudaError_t e = by_rows_first(R, first, [&](auto r, auto f) {
                return cudaFuncSetAttribute(sweep_kernel<decltype(r)::value, decltype(f)::value>,
                                            cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sweep_smem_bytes(gmax));
            });
            if (e != cudaSuccess) return e;
            e = by_rows_first(R, first, [&](auto r, auto f) {
                return cudaFuncSetAttribute(sweep_list_kernel<decltype(r)::value, decltype(f)::value>,
                                            cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sweep_smem_bytes(gmax));
            });
            if (e != cudaSuccess) return e;
        }
        cudaError_t e;
        if (R == kRowsSmall) {
            e = cudaFuncSetAttribute(inc_sweep_kernel<kRowsSmall, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)sweep_smem_bytes(gmax));
            if (e == cudaSuccess)
                e = cudaFuncSetAttribute(inc_sweep_kernel<kRowsSmall, true>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sweep_smem_bytes(gmax));
            if (e != cudaSuccess) return e;
        }
        e = by_rows(R, [&](auto r) {
            return cudaFuncSetAttribute(local_search_kernel<decltype(r)::value>,
                                        cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sweep_smem_bytes_ps(gmax));
        });
        if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
}

cudaError_t launch_sweep(const Geometry& g, const float2* P, const int* E, int n, const int2* tiles, int ntiles,
                         Slot* slot, int respect_done, unsigned long long* tilebest, int flags, cudaStream_t st)
{
    if (ntiles <= 0) return cudaSuccess;
    by_rows_first(g.rows, (flags & kSweepFirst) != 0, [&](auto r, auto f) {
        return launch_pdl(sweep_kernel<decltype(r)::value, decltype(f)::value>, dim3(ntiles), dim3(32 * g.warps),
                          sweep_smem_bytes(g), st, P, E, n, tiles, g.tj, slot, respect_done, tilebest, flags);
    });
    g_launches += 1;
    return cudaGetLastError();
}

cudaError_t launch_box_cull(const Geometry& g, const float2* P, const int* E, const int* G, int n, const int2* tiles,
                            int ntiles, Box* rbox, Box* cbox, int4* list, Slot* slot, int respect_done,
                            unsigned long long* tilebest, int flags, cudaStream_t st)
{
    const int TI = g.ti(), nrb = (n - 1 + TI - 1) / TI, ncc = (n + g.tj - 1) / g.tj;
    const int warps = nrb + ncc;
    const bool inc = (flags & kSweepIncremental) != 0;
    cudaError_t e = launch_pdl(box_kernel, dim3(std::min((warps + 7) / 8, TSP2OPT_BOX_BLOCKS)), dim3(256), 0, st, P, E, G, n, TI, nrb, g.tj, ncc,
                               rbox, cbox, slot, respect_done, inc && !(flags & kSweepFull) ? 1 : 0, 1);
    if (e != cudaSuccess) return e;
    e = launch_pdl(cull_kernel, dim3((ntiles + 256 * kCullPerThread - 1) / (256 * kCullPerThread)), dim3(256), 0, st,
                   tiles, ntiles, TI, g.tj, rbox, cbox, slot, list, tilebest, flags, respect_done, n, 1);
    g_launches += 2;
    return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_inc_sweep(const Geometry& g, const float2* P, const int* E, int n, const int2* tiles, int ntiles,
                             const int* tmap, int grid, Box* rbox, Box* cbox, Slot* slot, int respect_done,
                             unsigned long long* tilebest, int flags, cudaStream_t st)
{
    if (ntiles <= 0 || grid <= 0) return cudaSuccess;
    if (g.rows != kRowsSmall || g.warps != 1) return cudaErrorInvalidValue;  // instantiated for R = 7, one warp
    cudaError_t e = (flags & kSweepFirst)
                        ? launch_inc_sweep_t<kRowsSmall, true>(g, P, E, n, tiles, ntiles, tmap, grid, rbox, cbox, slot,
                                                               respect_done, tilebest, flags, st)
                        : launch_inc_sweep_t<kRowsSmall, false>(g, P, E, n, tiles, ntiles, tmap, grid, rbox, cbox,
                                                                slot, respect_done, tilebest, flags, st);
    g_launches += 1;
    return e != cudaSuccess ? e : cudaGetLastError();
}


cudaError_t launch_inc_ls(const Geometry& g, float2* P, int* E, int* tour, int n, const int2* tiles, int ntiles,
                          const int* tmap, Box* rbox, Box* cbox, Slot* slots, int parity, long long max_moves,
                          long long budget, int full, unsigned* bar, int* ctl, unsigned long long* tilebest, int flags,
                          unsigned long long* trace, long long trace_cap, int part_cols, cudaStream_t st)
{
    if (g.rows != kRowsSmall || g.warps != 1) return cudaErrorInvalidValue;
    int TI = g.ti(), TJ = g.tj, nrb = (n - 1 + TI - 1) / TI, ncc = (n + TJ - 1) / TJ;
    int tile_bytes = (int)((sweep_smem_bytes_ps(g) + 15) / 16 * 16);
    const size_t smem = (size_t)tile_bytes * (kIncLsThreads / 32);
    auto kern = (flags & kSweepFirst) ? inc_ls_kernel<kRowsSmall, true> : inc_ls_kernel<kRowsSmall, false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int per_sm = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kIncLsThreads, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) return cudaErrorInvalidConfiguration;
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int grid = sms;  // one CTA per SM (co-resident: cooperative launch)
    // kept tiles split into column parts over the CTA's warps (part_cols columns per part; 0: one warp
    // sweeps each whole kept tile)
    part_cols = std::min(std::max(part_cols, 0), TJ);
    if (flags & kSweepTileBounds) flags |= kSweepPartBounds;
    e = cudaMemsetAsync(bar, 0, 2 * sizeof(unsigned), st);  // count 0 (local_search_kernel leaves a counter)
    if (e != cudaSuccess) return e;
    void* args[] = {&P,     &E,    &tour,   &n,        &tiles,    &ntiles,    &tmap,   &TI,
                    &TJ,    &nrb,  &ncc,    &rbox,     &cbox,     &slots,     &parity, &max_moves,
                    &budget, &full, &bar,   &ctl,      &tilebest, &flags,     &trace,  &trace_cap,
                    &tile_bytes, &part_cols};
    g_launches += 1;
    return cudaLaunchCooperativeKernel((const void*)kern, dim3(grid), dim3(kIncLsThreads), args, smem, st);
}

size_t inc_ls2_ws_bytes(const Geometry& g, int n)
{
    const int TI = g.ti(), nrb = (n - 1 + TI - 1) / TI, ncc = (n + g.tj - 1) / g.tj;
    const int nsc = (ncc + kGroupChunks - 1) / kGroupChunks;
    return sizeof(unsigned long long) * (2 + (size_t)nrb * ncc + (size_t)nrb * nsc);
}

cudaError_t launch_inc_ls2(const Geometry& g, float2* P, int* E, int* tour, float2* P1, int* E1, int* T1, int n,
                           int np, const int* tmap, Box* rbox, Box* cbox, void* ws, Slot* slots, int parity,
                           long long max_moves, long long budget, int full, int* ctl, int flags,
                           unsigned long long* trace, long long trace_cap, int part_cols, int part_bound,
                           cudaStream_t st)
{
    if (g.rows != kRowsSmall || g.warps != 1) return cudaErrorInvalidValue;
    int TI = g.ti(), TJ = g.tj, nrb = (n - 1 + TI - 1) / TI, ncc = (n + TJ - 1) / TJ;
    int nsc = (ncc + kGroupChunks - 1) / kGroupChunks;
    unsigned long long* ctr = static_cast<unsigned long long*>(ws);
    unsigned long long* tb2 = ctr + 2;
    unsigned long long* sm2 = tb2 + (size_t)nrb * ncc;
    int tile_bytes = (int)((sweep_smem_bytes_ps(g) + 15) / 16 * 16);
    const size_t smem = (size_t)tile_bytes * kStageTiles;
    auto kern = (flags & kSweepFirst) ? inc_ls2_kernel<kRowsSmall, true> : inc_ls2_kernel<kRowsSmall, false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int per_sm = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kIncLsThreads, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) return cudaErrorInvalidConfiguration;
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    part_cols = part_cols > 0 ? std::min(part_cols, TJ) : kIncPartCols;
    if (part_bound && (flags & kSweepTileBounds)) flags |= kSweepPartBounds;
    e = cudaMemsetAsync(ctr, 0, sizeof(unsigned long long), st);  // the barrier's arrival counter
    if (e != cudaSuccess) return e;
    void* args[] = {&P,   &E,   &tour, &P1,    &E1,        &T1,    &n,       &np,        &tmap,
                    &TI,  &TJ,  &nrb,  &ncc,   &nsc,       &rbox,  &cbox,    &tb2,       &sm2,
                    &ctr, &slots, &parity, &max_moves, &budget, &full, &ctl, &flags, &trace,
                    &trace_cap, &tile_bytes, &part_cols};
    g_launches += 1;
    return cudaLaunchCooperativeKernel((const void*)kern, dim3(sms), dim3(kIncLsThreads), args, smem, st);
}

size_t inc_ls1_ws_bytes(const Geometry& g, int n)
{
    const int TI = g.ti(), nrb = (n - 1 + TI - 1) / TI, ncc = (n + g.tj - 1) / g.tj;
    const int nsc = (ncc + kGroupChunks - 1) / kGroupChunks;
    const size_t words = (4 + 4 + (size_t)nrb * ncc + (size_t)nrb * nsc + 3) / 4 * 4;  // boxes 32-byte aligned
    return sizeof(unsigned long long) * words + sizeof(Box) * 2 * ((size_t)nrb + ncc);
}

cudaError_t launch_inc_ls1(const Geometry& g, float2* P, int* E, int* tour, float2* P1, int* E1, int* T1, int n,
                           int np, const int* tmap, void* ws, Slot* slots, int parity, long long max_moves,
                           long long budget, int* ctl, int flags, unsigned long long* trace, long long trace_cap,
                           int part_cols, cudaStream_t st)
{
    if (g.rows != kRowsSmall || g.warps != 1) return cudaErrorInvalidValue;
    int TI = g.ti(), TJ = g.tj, nrb = (n - 1 + TI - 1) / TI, ncc = (n + TJ - 1) / TJ;
    int nsc = (ncc + kGroupChunks - 1) / kGroupChunks;
    unsigned long long* ctr = static_cast<unsigned long long*>(ws);
    unsigned long long* keys3 = ctr + 4;
    unsigned long long* tb2 = keys3 + 4;
    unsigned long long* sm2 = tb2 + (size_t)nrb * ncc;
    const size_t words = (4 + 4 + (size_t)nrb * ncc + (size_t)nrb * nsc + 3) / 4 * 4;  // Box is 32-byte aligned
    Box* rboxA = reinterpret_cast<Box*>(ctr + words);
    Box* cboxA = rboxA + nrb;
    Box* rboxB = cboxA + ncc;
    Box* cboxB = rboxB + nrb;
    int tile_bytes = (int)((sweep_smem_bytes_ps(g) + 15) / 16 * 16);
    const size_t smem = (size_t)tile_bytes * kStageTiles;
    auto kern = (flags & kSweepFirst) ? inc_ls1_kernel<kRowsSmall, true> : inc_ls1_kernel<kRowsSmall, false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int per_sm = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kIncLsThreads, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) return cudaErrorInvalidConfiguration;
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    // parts of a quarter tile, at least 4 columns (measured with one barrier: 8 of 32 columns, C5 MF 17.4
    // vs 18.3 us per move with 4; profiles/r02_exp_inc_parts.jsonl)
    part_cols = part_cols > 0 ? std::min(part_cols, TJ) : std::max(kIncPartCols, TJ / 4);
    e = cudaMemsetAsync(ctr, 0, sizeof(unsigned long long), st);
    if (e != cudaSuccess) return e;
    void* args[] = {&P,     &E,     &tour,  &P1,    &E1,       &T1,    &n,      &np,        &tmap,   &TI,
                    &TJ,    &nrb,   &ncc,   &nsc,   &rboxA,    &cboxA, &rboxB,  &cboxB,     &tb2,    &sm2,
                    &ctr,   &keys3, &slots, &parity, &max_moves, &budget, &ctl,  &flags,     &trace,  &trace_cap,
                    &tile_bytes, &part_cols};
    g_launches += 1;
    return cudaLaunchCooperativeKernel((const void*)kern, dim3(sms), dim3(kIncLsThreads), args, smem, st);
}

cudaError_t launch_dense_ls(const Geometry& g, float2* P, int* E, int* tour, int n, const int2* tiles, int ntiles,
                            Slot* slots, int parity, long long max_moves, long long budget, unsigned* bar, int* ctl,
                            int flags, unsigned long long* tilebest, unsigned long long* trace, long long trace_cap,
                            cudaStream_t st)
{
    if (g.warps != 1) return cudaErrorInvalidValue;
    int TJ = g.tj;
    int tile_bytes = (int)((sweep_smem_bytes_ps(g) + 15) / 16 * 16);
    const size_t smem = (size_t)tile_bytes * (kIncLsThreads / 32);
    auto kern = g.rows == kRowsSmall ? dense_ls_kernel<kRowsSmall> : dense_ls_kernel<kRowsLarge>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int per_sm = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kIncLsThreads, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) return cudaErrorInvalidConfiguration;
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    e = cudaMemsetAsync(bar, 0, 2 * sizeof(unsigned), st);  // count 0 (local_search_kernel leaves a counter)
    if (e != cudaSuccess) return e;
    void* args[] = {&P, &E, &tour, &n, &tiles, &ntiles, &TJ, &slots, &parity, &max_moves, &budget, &bar, &ctl,
                    &flags, &tilebest, &trace, &trace_cap, &tile_bytes};
    g_launches += 1;
    return cudaLaunchCooperativeKernel((const void*)kern, dim3(sms), dim3(kIncLsThreads), args, smem, st);
}

int inc_sweep_grid(const Geometry& g)
{
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, inc_sweep_kernel<kRowsSmall, false>, 32,
                                                      sweep_smem_bytes(g)) != cudaSuccess)
        return 0;
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    return per_sm * sms;
}

int sweep_list_grid(const Geometry& g, int ntiles)
{
    int per_sm = 0;
    cudaError_t e = by_rows(g.rows, [&](auto r) {
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, sweep_list_kernel<decltype(r)::value, false>,
                                                             32 * g.warps, sweep_smem_bytes(g));
    });
    if (e != cudaSuccess) return 0;
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int grid = per_sm * sms;
    return grid < ntiles ? grid : ntiles;
}

cudaError_t launch_cull_sweep(const Geometry& g, const float2* P, const int* E, int n, const int2* tiles,
                              int ntiles, int grid, Box* rbox, Box* cbox, int4* list, Slot* slot, int respect_done,
                              unsigned long long* tilebest, int flags, cudaStream_t st)
{
    if (ntiles <= 0 || grid <= 0) return cudaSuccess;
    const int TI = g.ti(), nrb = (n - 1 + TI - 1) / TI, ncc = (n + g.tj - 1) / g.tj;
    const int warps = nrb + ncc;
    const bool inc = (flags & kSweepIncremental) != 0;
    cudaError_t e = launch_pdl(box_kernel, dim3(std::min((warps + 7) / 8, TSP2OPT_BOX_BLOCKS)), dim3(256), 0, st, P, E, (const int*)nullptr, n, TI,
                               nrb, g.tj, ncc, rbox, cbox, slot, respect_done, inc && !(flags & kSweepFull) ? 1 : 0, 0);
    if (e != cudaSuccess) return e;
    e = launch_pdl(cull_kernel, dim3((ntiles + 256 * kCullPerThread - 1) / (256 * kCullPerThread)), dim3(256), 0, st,
                   tiles, ntiles, TI, g.tj, rbox, cbox, slot, list, tilebest, flags, respect_done, n, 0);
    if (e != cudaSuccess) return e;
    if (inc) flags = (flags | kSweepLocal) & ~kSweepSeed;  // tile-local minima, reusable while clean
    e = by_rows_first(g.rows, (flags & kSweepFirst) != 0, [&](auto r, auto f) {
        return launch_pdl(sweep_list_kernel<decltype(r)::value, decltype(f)::value>, dim3(grid), dim3(32 * g.warps),
                          sweep_smem_bytes(g), st, P, E, n, tiles, list, g.tj, slot, respect_done, tilebest, flags);
    });
    g_launches += 3;
    if (e != cudaSuccess) return e;
    return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_apply(float2* P, int* E, int* tour, int n, const Slot* in, Slot* out, long long max_moves,
                         int explicit_move, int ei, int ej, unsigned long long* trace, long long trace_cap,
                         int* pos, cudaStream_t st)
{
    int blocks = (n / 2 + 255) / 256;
    if (blocks < 1) blocks = 1;
    if (blocks > 4 * 148) blocks = 4 * 148;
    cudaError_t e = launch_pdl(apply_kernel, dim3(blocks), dim3(256), 0, st, P, E, tour, in, out, max_moves,
                               explicit_move, ei, ej, trace, trace_cap, pos);
    if (e != cudaSuccess) return e;
    g_launches += 1;
    return cudaGetLastError();
}

int local_search_grid(const Geometry& g, int ntiles)
{
    int per_sm = 0;
    cudaError_t e = by_rows(g.rows, [&](auto r) {
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, local_search_kernel<decltype(r)::value>,
                                                             32 * g.warps, sweep_smem_bytes_ps(g));
    });
    if (e != cudaSuccess) return 0;
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int grid = per_sm * sms;
    return grid < ntiles ? grid : ntiles;
}

cudaError_t launch_local_search(const Geometry& g, float2* P, int* E, int* tour, int n, const int2* tiles, int ntiles,
                                Slot* slots, int parity, long long max_moves, long long budget, unsigned* bar,
                                int* ctl, unsigned long long* tilebest, int flags, unsigned long long* trace,
                                long long trace_cap, cudaStream_t st)
{
    int grid = local_search_grid(g, ntiles);
    if (grid < 1) return cudaErrorInvalidConfiguration;
    int TJ = g.tj;
    // the barrier's arrival counter (the other persistent kernels' (count, generation) pair reads as
    // count 0 after this as well)
    cudaError_t e = cudaMemsetAsync(bar, 0, 2 * sizeof(unsigned), st);
    if (e != cudaSuccess) return e;
    void* args[] = {&P, &E, &tour, &n, &tiles, &ntiles, &TJ, &slots, &parity, &max_moves, &budget, &bar, &ctl,
                    &tilebest, &flags, &trace, &trace_cap};
    g_launches += 1;
    return by_rows(g.rows, [&](auto r) {
        return cudaLaunchCooperativeKernel((const void*)local_search_kernel<decltype(r)::value>, dim3(grid),
                                           dim3(32 * g.warps), args, sweep_smem_bytes_ps(g), st);
    });
}

cudaError_t run_selftest_sqrt(double* max_rel, int* zero_ok)
{
    unsigned* d = nullptr;
    cudaError_t err = cudaMalloc(&d, 2 * sizeof(unsigned));
    if (err != cudaSuccess) return err;
    cudaMemset(d, 0, 2 * sizeof(unsigned));
    selftest_sqrt_kernel<<<148 * 8, 256>>>(d, d + 1);
    g_launches += 1;
    unsigned h[2] = {0, 0};
    err = cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    cudaFree(d);
    float f;
    memcpy(&f, &h[0], sizeof(f));
    *max_rel = f;
    *zero_ok = h[1] == 0;
    return err;
}

cudaError_t read_phases(long long* out16, int reset)
{
#ifdef TSP2OPT_PHASE_TIMING
    unsigned long long ph[16];
    cudaError_t ep = cudaMemcpyFromSymbol(ph, g_phase, sizeof(ph));
    if (ep != cudaSuccess) return ep;
    for (int k = 0; k < 16; k++) out16[k] = (long long)ph[k];
    if (reset) {
        const unsigned long long z[16] = {};
        ep = cudaMemcpyToSymbol(g_phase, z, sizeof(z));
    }
    return ep;
#else
    (void)reset;
    for (int k = 0; k < 16; k++) out16[k] = -1;
    return cudaSuccess;
#endif
}

cudaError_t read_stats(long long* out4, int reset)
{
#if defined(TSP2OPT_STATS) || defined(TSP2OPT_TILE_TIMING)
    unsigned long long h[4];
    cudaError_t e = cudaMemcpyFromSymbol(h, g_stats, sizeof(h));
    if (e != cudaSuccess) return e;
    for (int k = 0; k < 4; k++) out4[k] = (long long)h[k];
    if (reset) {
        const unsigned long long z[4] = {0, 0, 0, 0};
        e = cudaMemcpyToSymbol(g_stats, z, sizeof(z));
    }
    return e;
#else
    (void)reset;
    for (int k = 0; k < 4; k++) out4[k] = -1;
    return cudaSuccess;
#endif
}

cudaError_t run_selftest(long long* out4)
{
    unsigned long long* d = nullptr;
    cudaError_t err = cudaMalloc(&d, 4 * sizeof(unsigned long long));
    if (err != cudaSuccess) return err;
    unsigned long long init[4] = {0, 0, ~0ULL, ~0ULL};
    cudaMemcpy(d, init, sizeof(init), cudaMemcpyHostToDevice);
    selftest_dist_kernel<<<148 * 8, 256>>>(2LL * 32767 * 32767, d, d + 2);
    selftest_filter_kernel<<<148 * 8, 256>>>(d + 1, d + 3);
    g_launches += 2;
    unsigned long long h[4];
    err = cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    cudaFree(d);
    for (int k = 0; k < 4; k++) out4[k] = (long long)h[k];
    return err;
}

}  // namespace tsp2opt
