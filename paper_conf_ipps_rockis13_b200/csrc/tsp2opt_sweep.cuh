// tsp2opt_sweep.cuh -- the sweep of one (row block x column chunk) tile
// (SURVEY.md §8(a) rows a4 + a5), shared by the per-sweep kernel and the
// persistent local-search kernel of tsp2opt_kernels.cu.
//
// One CTA = one tile = rows [I0, I0 + 32*R*NW) x columns [J0, J0 + TJ) -- the
// paper's problem division into "2 coordinate ranges" (L18 §IV.B; L20 Fig. 7,
// Listing 2 "2 sets of coordinates needed, A for point i and B for point j").
// Each lane owns R consecutive rows (R+1 cities in registers, packed FP32x2);
// the warp walks the tile's columns, column city j being a shared-memory
// broadcast.  Per column step the lane computes the R+1 squared distances of
// its rows to column j+1 (diagonal reuse: s(i+1, j+1) of pair (i, j) is
// s(i', j') of pair (i', j') = (i+1, j+1)) and tests every pair (i, j) with
// the exact necessary condition of DESIGN.md §5.2:
//     delta(i,j) <= B - 1   ==>   D(i,j) <= e_i + a1   or   D(i+1,j+1) <= e_j + a2
// (a1 + a2 = B - 2) on squared distances (no sqrt).  Pairs that pass are
// evaluated exactly (integer nint, the oracle's arithmetic) and accepted iff
// delta < B; B is the lane's running bound, started from the global best.
// Pairs are visited in increasing Fig. 3 cell order per lane, so a strict '<'
// keeps the lowest cell among equal deltas (reading R5).
//
// PS (persistent) selects the global-load flavour: the per-sweep kernel reads
// P and E through the read-only path (__ldg); the persistent kernel rewrites P
// and E between sweeps, so it uses plain coherent loads (L1 is invalidated by
// the gpu-scope fence of its grid barrier).
#pragma once

#include "tsp2opt_device.cuh"

namespace tsp2opt {

#if defined(TSP2OPT_STATS) || defined(TSP2OPT_TILE_TIMING)
// Instrumented builds only (TSP2OPT_TILE_TIMING: [0] prologue cycles -- loads, staging,
// the seed key --, [1] walk cycles, [2] tiles walked, [3] the slowest tile's cycles): [0] warp column steps, [1] steps taking the exact
// path, [2] candidate pairs evaluated exactly, [3] warp tiles walked (not
// skipped by the tile bound).
__device__ unsigned long long g_stats[4];
#endif

template <bool PS, typename T>
__device__ __forceinline__ T gld(const T* p)
{
    if constexpr (PS) return *p;
    else return __ldg(p);
}

template <int R>
struct Rows {
    float2 xp[(R + 1) / 2];  // (x_r, x_{r+1}) packed pairs, biased floats, r = 0..R
    float2 yp[(R + 1) / 2];
};

template <int R>
__device__ __forceinline__ void column_sq(float (&s)[R + 1], const Rows<R>& rows, float4 c)
{
    const float2 ncx = make_float2(c.x, c.y), ncy = make_float2(c.z, c.w);
#pragma unroll
    for (int q = 0; q < (R + 1) / 2; q++) {
        float2 v = sq2(rows.xp[q], rows.yp[q], ncx, ncy);
        s[2 * q] = v.x;
        s[2 * q + 1] = v.y;
    }
}

template <int R>
struct Bound {
    int B;          // accept delta < B (lane-local running bound)
    float Bf;       // B as float (exact)
    float a2f;      // column offset a2 = (B - 2) - a1
    int a2;
    float srow[R];  // row thresholds: D(i_r, j) <= e_{i_r} + a1  <=>  s <= srow[r]
};

// Thresholds of the exact necessary condition for bound B:
// delta <= B - 1 = c  ==>  D(i,j) <= e_i + a1  or  D(i+1,j+1) <= e_j + a2,
// a1 = floor((c - 1) / 2), a2 = c - 1 - a1.
// Row edges are floats (exact integers): no int <-> float conversions (XU
// pipe) when the bound drops mid-tile.
template <int R>
__device__ __forceinline__ void set_bound(Bound<R>& b, const float* erowf, int B)
{
    b.B = B;
    b.Bf = (float)B;
    const int c = B - 1;
    const int a1 = (c - 1) >> 1;
    const int a2 = c - 1 - a1;
    b.a2f = (float)a2;
    b.a2 = a2;
    const float a1f = (float)a1;
#pragma unroll
    for (int r = 0; r < R; r++) b.srow[r] = sq_threshold(erowf[r] + a1f);
}

// Shared memory of one tile: the column chunk (the paper's coordinate range
// "B", L20 Listing 2) and the edges of the CTA's rows (range "A").
constexpr int kMaxWarpsPerTile = 4;

// One staged column c = j - J0 is a record of kColRec float4 (48 bytes):
//   [0] (-x, -x, -y, -y)  biased floats, negated
//   [1] (e_j, thr_0, thr_1, thr_2), [2] (thr_3, -, -, -)
// thr_w = sq_threshold(e_j + a2w) is warp w's column threshold (fill_colthr).
// Interleaving them lets the walk step ONE shared-memory pointer per column
// (immediate offsets for xy, the next column and the threshold).
constexpr int kColRec = 3;

struct TileSmem {
    float4* col;   // [TJ + 2] column records: columns J0..J1 and one spare
    float* rowe;   // [TI = 32 * R * warps]: e_i of the CTA's rows, as float
    float2* rowp;  // [32 * warps * (R + 1)]: each lane's R + 1 row cities (biased), for the rare path --
                   // shared memory, not a reload of P that may miss L1 (persistent kernels invalidate it)
    __device__ TileSmem(void* base, int TJ, int TI)
        : col(reinterpret_cast<float4*>(base)),
          rowe(reinterpret_cast<float*>(col + kColRec * (TJ + 2))),
          rowp(reinterpret_cast<float2*>(rowe + TI))
    {
    }
    __device__ float4 xy(int c) const { return col[kColRec * c]; }
    __device__ float e(int c) const { return reinterpret_cast<const float*>(col + kColRec * c + 1)[0]; }
    __device__ void put(int c, float2 p, float e) const
    {
        col[kColRec * c] = make_float4(-p.x, -p.x, -p.y, -p.y);
        reinterpret_cast<float*>(col + kColRec * c + 1)[0] = e;
    }
};

// Column record accessors for a walk's running pointer (rec = &col[kColRec * c]).
__device__ __forceinline__ float rec_e(const float4* rec) { return reinterpret_cast<const float*>(rec + 1)[0]; }
__device__ __forceinline__ float rec_thr(const float4* rec, int w) { return reinterpret_cast<const float*>(rec + 1)[1 + w]; }

// Same as set_bound, from the lane's row edges in shared memory (rare: the
// bound dropped mid-tile).
template <int R>
__device__ __forceinline__ void reset_bound(Bound<R>& b, const float* my_rowe, int B)
{
    set_bound<R>(b, my_rowe, B);
}

// The fast test of one column step: does any pair (i_r, j), r < R, of this
// lane pass the necessary condition?  Four independent predicate chains keep
// the dependency depth short.
template <int R, bool MASK>
__device__ __forceinline__ bool step_any(const Bound<R>& b, const float (&cur)[R + 1], const float (&nxt)[R + 1],
                                         float scol, int row0, int j)
{
    if (!MASK) {
        float m = nxt[1];
#pragma unroll
        for (int r = 2; r <= R; r++) m = fminf(m, nxt[r]);
        bool a0 = m <= scol, a1 = false, a2 = false, a3 = false;
#pragma unroll
        for (int r = 0; r < R; r++) {
#ifndef TSP2OPT_ROWTEST_FLOAT
            // cur >= +0 and srow is either >= +0 or negative (t < 0, sq_threshold), so the
            // signed integer order of the IEEE bits equals the float order here (ISETP and
            // FSETP share the ALU pipe's half rate; measured 1 % faster, r02_exp_sweep.jsonl)
            const bool t = __float_as_int(cur[r]) <= __float_as_int(b.srow[r]);
#else
            const bool t = cur[r] <= b.srow[r];
#endif
            if ((r & 3) == 0) a0 |= t;
            else if ((r & 3) == 1) a1 |= t;
            else if ((r & 3) == 2) a2 |= t;
            else a3 |= t;
        }
        return (a0 | a1) | (a2 | a3);
    } else {
        bool any = false;
#pragma unroll
        for (int r = 0; r < R; r++) any |= ((cur[r] <= b.srow[r]) || (nxt[r + 1] <= scol)) && (row0 + r < j);
        return any;
    }
}

// Exact evaluation of this lane's candidate pairs of column step j (rare path;
// only lanes with a candidate run it).  A second, tighter necessary condition
// is applied first: nint(sqrt(s)) >= sqrt(s) - 1/2, so
//     delta <= B - 1  ==>  sqrt(s1) + sqrt(s2) <= e_i + e_j + B,
// evaluated with MUFU.SQRT on the float squared distances already in
// registers; its error (< 0.04, the sqrt error is bounded
// exhaustively by tsp2opt_selftest) is covered by a 0.5 slack.  Survivors are
// evaluated with integer nint distances -- the oracle's arithmetic -- and
// accepted iff delta < B, in increasing cell order.

template <int R, bool MASK, bool PS, bool FIRST>
__device__ __forceinline__ void exact_step(Bound<R>& b, const float (&cur)[R + 1], const float (&nxt)[R + 1],
                                           float scol, int row0, int j, float4 c0, float4 c1, float ej,
                                           const float* my_rowe, const float2* my_rowp, unsigned long long& mykey)
{
    const float lim = ej + b.Bf + 0.5f;
    unsigned mask = 0;
#pragma unroll
    for (int r = 0; r < R; r++) {
        bool cand = (cur[r] <= b.srow[r]) || (nxt[r + 1] <= scol);
        if (MASK) cand = cand && (row0 + r < j);
        if (cand) cand = sqrt_approx(cur[r]) + sqrt_approx(nxt[r + 1]) <= my_rowe[r] + lim;
        mask |= (cand ? 1u : 0u) << r;
    }
#ifdef TSP2OPT_STATS
    atomicAdd(&g_stats[2], (unsigned long long)__popc(mask));
#endif
    if (!mask) return;
    const int xj = unbias(-c0.x), yj = unbias(-c0.z);
    const int xj1 = unbias(-c1.x), yj1 = unbias(-c1.z);
    float Bf = b.Bf;
    while (mask) {  // ascending r == ascending cell number
        const int r = __ffs(mask) - 1;
        mask &= mask - 1;
        // PS (persistent kernels): the row cities staged in shared memory (P's L1 lines are
        // invalidated by every grid barrier); otherwise my_rowp = P + row0, read through L1
        const float2 pi = PS ? my_rowp[r] : __ldg(my_rowp + r), pi1 = PS ? my_rowp[r + 1] : __ldg(my_rowp + r + 1);
        // nint from the float path when it is unambiguous: |sqrt_approx(s_f) - sqrt(s)|
        // < 0.03, so |r - m| < 0.45 for the nearest integer m
        // proves nint(sqrt(s)) == m.  Otherwise the integer nint (rare).
        const float dx = pi.x + c0.x, dy = pi.y + c0.z, dx1 = pi1.x + c1.x, dy1 = pi1.y + c1.z;  // exact
        float d1, d2;
        if (!nint_from_float(fmaf(dx, dx, dy * dy), d1))
            d1 = (float)exact_dist_xy(unbias(pi.x), unbias(pi.y), xj, yj);
        if (!nint_from_float(fmaf(dx1, dx1, dy1 * dy1), d2))
            d2 = (float)exact_dist_xy(unbias(pi1.x), unbias(pi1.y), xj1, yj1);
        const float d = (d1 + d2) - (my_rowe[r] + ej);  // exact: integers < 2^24
        if (FIRST) {
            // first improvement (reading R20): the lane's first improving pair is its
            // lowest cell; the key's delta is the marker kFirstDelta (resolved later)
            if (d < 0.0f && mykey == kKeyNone) mykey = pack_key(kFirstDelta, row0 + r, j);
            continue;
        }
        if (d < Bf) {
            Bf = d;
            mykey = pack_key((int)d, row0 + r, j);
        }
    }
    if (!FIRST && Bf < b.Bf) {
        b.B = (int)Bf;
        b.Bf = Bf;
    }
}

// The column thresholds of this warp's walk, thr_w of columns rec[0 .. count)
// = sq_threshold(e_j + a2w) with a2w the largest column offset a2 of the
// warp's lanes: a larger a2 only weakens each lane's necessary condition (its
// own a1 + a2 >= c - 1 still holds), so one threshold per column serves the
// whole warp.  Written when the walk starts and again after a lane's bound
// dropped (rare); it saves the walk four FP32 instructions per column step.
// Returns a2w.
__device__ __forceinline__ int fill_colthr(int a2, float4* rec, int w, int count)
{
    const int a2w = __reduce_max_sync(0xffffffffu, a2);
    const float a2wf = (float)a2w;
    for (int k = (int)(threadIdx.x & 31); k < count; k += 32) {
        float* r = reinterpret_cast<float*>(rec + kColRec * k + 1);
        r[1 + w] = sq_threshold(r[0] + a2wf);
    }
    __syncwarp();
    return a2w;
}

// One column step of the walk at column j, rec = its record.  Returns true
// (FIRST only) once some lane of the warp holds an improving pair: every later
// column has higher cell numbers, so the walk can stop.  left = columns from j
// to the end of the chunk.
template <int R, bool MASK, bool PS, bool FIRST>
__device__ __forceinline__ bool column_step(const Rows<R>& rows, Bound<R>& b, const float (&cur)[R + 1],
                                            float (&nxt)[R + 1], int row0, int j, float4* rec, int w, int left,
                                            int& a2w, const float* my_rowe, const float2* my_rowp,
                                            unsigned long long& mykey)
{
    const float4 c1 = rec[kColRec];
    column_sq<R>(nxt, rows, c1);
    const float scol = rec_thr(rec, w);
    const bool any = step_any<R, MASK>(b, cur, nxt, scol, row0, j);
#ifdef TSP2OPT_STATS
    if ((threadIdx.x & 31) == 0) atomicAdd(&g_stats[0], 1ULL);
#endif
    if (__builtin_expect(__any_sync(0xffffffffu, any), 0)) {
#ifdef TSP2OPT_STATS
        if ((threadIdx.x & 31) == 0) atomicAdd(&g_stats[1], 1ULL);
#endif
        const int B0 = b.B;
        if (any) exact_step<R, MASK, PS, FIRST>(b, cur, nxt, scol, row0, j, rec[0], c1, rec_e(rec), my_rowe, my_rowp,
                                                mykey);
        if (FIRST) return __any_sync(0xffffffffu, mykey != kKeyNone);
        // share the warp's best: a lane may accept delta <= (best of another lane)
        const int wb = __reduce_min_sync(0xffffffffu, b.B);
        const int nb = min(b.B, wb + 1);
        if (nb < B0) reset_bound<R>(b, my_rowe, nb);
        if (__reduce_max_sync(0xffffffffu, b.a2) != a2w) a2w = fill_colthr(b.a2, rec + kColRec, w, left - 1);
    }
    return false;
}

// The rare path of column step j for the grouped walk below: the step's
// squared distances are recomputed from the lane's rows and the column records
// (the walk's arrays have moved on), then exactly as column_step's rare branch.
template <int R, bool MASK, bool PS, bool FIRST>
__device__ __forceinline__ bool rare_step(const Rows<R>& rows, Bound<R>& b, int row0, int j, float4* rec, int w,
                                          int left, int& a2w, const float* my_rowe, const float2* my_rowp,
                                          unsigned long long& mykey)
{
    float cur[R + 1], nxt[R + 1];
    column_sq<R>(cur, rows, rec[0]);
    const float4 c1 = rec[kColRec];
    column_sq<R>(nxt, rows, c1);
    const float scol = rec_thr(rec, w);
    const bool any = step_any<R, MASK>(b, cur, nxt, scol, row0, j);
    if (!__any_sync(0xffffffffu, any)) return false;
#ifdef TSP2OPT_STATS
    if ((threadIdx.x & 31) == 0) atomicAdd(&g_stats[1], 1ULL);
#endif
    const int B0 = b.B;
    if (any) exact_step<R, MASK, PS, FIRST>(b, cur, nxt, scol, row0, j, rec[0], c1, rec_e(rec), my_rowe, my_rowp, mykey);
    if (FIRST) return __any_sync(0xffffffffu, mykey != kKeyNone);
    const int wb = __reduce_min_sync(0xffffffffu, b.B);
    const int nb = min(b.B, wb + 1);
    if (nb < B0) reset_bound<R>(b, my_rowe, nb);
    if (__reduce_max_sync(0xffffffffu, b.a2) != a2w) a2w = fill_colthr(b.a2, rec + kColRec, w, left - 1);
    return false;
}

#ifndef TSP2OPT_VOTE_STEPS
#define TSP2OPT_VOTE_STEPS 1  // column steps per warp vote (even, or 1 = a vote every step; measured: 2 and 4
                              // are 6 % and 8 % slower at C5, profiles/r02_exp_sweep.jsonl)
#endif

template <int R, bool MASK, bool PS, bool FIRST>
__device__ __forceinline__ void walk(const Rows<R>& rows, Bound<R>& b, int row0, int jstart, int J0, int J1,
                                     const TileSmem& sm, const float* my_rowe, const float2* my_rowp,
                                     unsigned long long& mykey, int w)
{
    float4* rec = sm.col + kColRec * (jstart - J0);
    int a2w = fill_colthr(b.a2, rec, w, J1 - jstart);
    float sa[R + 1], sb[R + 1];
    column_sq<R>(sa, rows, rec[0]);
    int j = jstart;
    constexpr int V = TSP2OPT_VOTE_STEPS;
    static_assert(V == 1 || V % 2 == 0, "grouped steps keep sa as the next group's current column");
    if constexpr (V > 1) {
        // V column steps per warp vote: one straight-line region of V steps for the
        // scheduler and one VOTE + branch per group; a group with a candidate re-runs
        // its steps one by one on the rare path (rare_step), in increasing cell order.
        for (; j + V <= J1; j += V, rec += V * kColRec) {
            bool any = false;
#pragma unroll
            for (int v = 0; v < V; v++) {
                float(&cur)[R + 1] = (v & 1) ? sb : sa;
                float(&nxt)[R + 1] = (v & 1) ? sa : sb;
                column_sq<R>(nxt, rows, rec[(v + 1) * kColRec]);
                any |= step_any<R, MASK>(b, cur, nxt, rec_thr(rec + v * kColRec, w), row0, j + v);
            }
#ifdef TSP2OPT_STATS
            if ((threadIdx.x & 31) == 0) atomicAdd(&g_stats[0], (unsigned long long)V);
#endif
            if (__builtin_expect(__any_sync(0xffffffffu, any), 0)) {
#pragma unroll 1
                for (int v = 0; v < V; v++)
                    if (rare_step<R, MASK, PS, FIRST>(rows, b, row0, j + v, rec + v * kColRec, w, J1 - j - v, a2w,
                                                      my_rowe, my_rowp, mykey))
                        return;
                column_sq<R>(sa, rows, rec[V * kColRec]);  // the next group's current column
            }
        }
    }
    for (; j + 1 < J1; j += 2, rec += 2 * kColRec) {
        if (column_step<R, MASK, PS, FIRST>(rows, b, sa, sb, row0, j, rec, w, J1 - j, a2w, my_rowe, my_rowp, mykey))
            return;
        if (column_step<R, MASK, PS, FIRST>(rows, b, sb, sa, row0, j + 1, rec + kColRec, w, J1 - j - 1, a2w, my_rowe,
                                            my_rowp, mykey))
            return;
    }
    if (j < J1)
        column_step<R, MASK, PS, FIRST>(rows, b, sa, sb, row0, j, rec, w, J1 - j, a2w, my_rowe, my_rowp, mykey);
}

// Tile-level form of the same exact necessary condition (a bound on all of the
// tile's pairs at once).  Every squared distance the walk would compare is
// between a city of the warp's row block (rows r = 0..R of every lane) and a
// column city c in [cbeg, cend] of the staged chunk, so it is at least the
// squared distance d2 between the two bounding boxes; every threshold it is
// compared with is at most max(max_r srow[r], sq_threshold(max_j e_j + a2)).
// If d2 exceeds that (with 2^-20 slack for the float roundings of d2 and of
// the walk's own s_f >= s (1 - 2^-23)), no pair of the tile can pass the
// per-pair filter and the walk is skipped.  Spatially coherent tours (the
// later sweeps of a local search) skip most tiles; random tours skip none.
template <int R>
__device__ __forceinline__ bool tile_may_pass(const Rows<R>& rows, const Bound<R>& b, const TileSmem& sm, int cbeg,
                                              int cend)
{
    float xlo = rows.xp[0].x, xhi = xlo, ylo = rows.yp[0].x, yhi = ylo;
#pragma unroll
    for (int q = 0; q < (R + 1) / 2; q++) {
        xlo = fminf(xlo, fminf(rows.xp[q].x, rows.xp[q].y));
        xhi = fmaxf(xhi, fmaxf(rows.xp[q].x, rows.xp[q].y));
        ylo = fminf(ylo, fminf(rows.yp[q].x, rows.yp[q].y));
        yhi = fmaxf(yhi, fmaxf(rows.yp[q].x, rows.yp[q].y));
    }
    float smax = b.srow[0];
#pragma unroll
    for (int r = 1; r < R; r++) smax = fmaxf(smax, b.srow[r]);
    // column cities are staged negated: colxy = (-x, -x, -y, -y)
    float cxlo = 3.0e38f, cxhi = -3.0e38f, cylo = 3.0e38f, cyhi = -3.0e38f, emax = -1.0f;
    for (int c = cbeg + (int)(threadIdx.x & 31); c <= cend; c += 32) {
        const float4 v = sm.xy(c);
        cxlo = fminf(cxlo, -v.x);
        cxhi = fmaxf(cxhi, -v.x);
        cylo = fminf(cylo, -v.z);
        cyhi = fmaxf(cyhi, -v.z);
        if (c < cend) emax = fmaxf(emax, sm.e(c));  // e_j of the step's own column j < J1
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        xlo = fminf(xlo, __shfl_xor_sync(0xffffffffu, xlo, o));
        xhi = fmaxf(xhi, __shfl_xor_sync(0xffffffffu, xhi, o));
        ylo = fminf(ylo, __shfl_xor_sync(0xffffffffu, ylo, o));
        yhi = fmaxf(yhi, __shfl_xor_sync(0xffffffffu, yhi, o));
        smax = fmaxf(smax, __shfl_xor_sync(0xffffffffu, smax, o));
        cxlo = fminf(cxlo, __shfl_xor_sync(0xffffffffu, cxlo, o));
        cxhi = fmaxf(cxhi, __shfl_xor_sync(0xffffffffu, cxhi, o));
        cylo = fminf(cylo, __shfl_xor_sync(0xffffffffu, cylo, o));
        cyhi = fmaxf(cyhi, __shfl_xor_sync(0xffffffffu, cyhi, o));
        emax = fmaxf(emax, __shfl_xor_sync(0xffffffffu, emax, o));
    }
    const float thr = fmaxf(smax, sq_threshold(emax + b.a2f));
    // box gaps: differences of biased floats are exact integers
    const float gx = fmaxf(0.f, fmaxf(cxlo - xhi, xlo - cxhi));
    const float gy = fmaxf(0.f, fmaxf(cylo - yhi, ylo - cyhi));
    const float d2 = fmaf(gx, gx, gy * gy);
    return d2 * 0.99999904632568359375f <= thr;  // (1 - 2^-20)
}

// Shared memory bytes of a tile with TJ columns and TI rows; rowp: the
// persistent kernels' staged row cities, (TI / R) * (R + 1) <= TI + TI / 7
// entries for R >= 7, plus slack.
__host__ __device__ inline size_t tile_smem_bytes(int TJ, int TI, bool rowp = false)
{
    return (size_t)(TJ + 2) * kColRec * sizeof(float4) + (size_t)TI * sizeof(float) +
           (rowp ? (size_t)(TI + TI / 7 + 32) * sizeof(float2) : 0);
}

// One tile.  All global loads of the tile (the lane's rows and row edges, the
// CTA's share of the column chunk, the global best key) are issued before the
// first use so their latencies overlap; then the column chunk and the row
// edges are staged in shared memory, every warp walks the chunk, and the warp
// minima are published with one atomicMin each (L16 Fig. 4 "Get best local
// pair ... Get best global pair"; min is order-independent, so the result is
// deterministic).  The caller synchronises the CTA before reusing `sm`.

//
// WT (warp tile): the tile belongs to ONE warp with its own TileSmem (the
// persistent incremental local search, where each warp of a large CTA sweeps
// its own tiles); warp synchronisation instead of block barriers.
template <int R, bool PS, bool FIRST = false, bool WT = false>
__device__ __forceinline__ void sweep_tile(const float2* P, const int* E, int n, int2 tile, int TJ, Slot* slot,
                                           const TileSmem& sm, unsigned long long* tilebest, int flags)
{
#ifdef TSP2OPT_TILE_TIMING
    const long long tt0 = clock64();
#endif
    const int I0 = tile.x, J0 = tile.y;
    const int J1 = min(J0 + TJ, n);  // columns j in [J0, J1), j <= n-1
    const int ncol = J1 - J0;
    const int warp = WT ? 0 : threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int tid = WT ? lane : threadIdx.x, nthr = WT ? 32 : blockDim.x;
    const int wrow0 = I0 + warp * 32 * R;
    const int row0 = wrow0 + lane * R;
    const int jstart = max(J0, wrow0 + 1);  // no pair of this warp has j <= wrow0
    const bool active = jstart < J1;        // warp-uniform
    float* my_rowe = sm.rowe + tid * R;  // stride R (odd): conflict-free
    float2* my_rowp = PS ? sm.rowp + tid * (R + 1) : const_cast<float2*>(P) + row0;

    Rows<R> rows;
    float erow[R];
    if (active) {
#pragma unroll
        for (int q = 0; q < (R + 1) / 2; q++) {
            const float2 p0 = gld<PS>(P + row0 + 2 * q), p1 = gld<PS>(P + row0 + 2 * q + 1);
            rows.xp[q] = make_float2(p0.x, p1.x);
            rows.yp[q] = make_float2(p0.y, p1.y);
            if (PS) {
                my_rowp[2 * q] = p0;
                my_rowp[2 * q + 1] = p1;
            }
        }
#pragma unroll
        for (int r = 0; r < R; r++) erow[r] = (float)gld<PS>(E + row0 + r);
    }
    for (int c = tid; c <= ncol + 1; c += nthr) {  // J1 <= n: P[n] = P[0]; + 1 spare column
        const float2 p = gld<PS>(P + J0 + c);
        const int e = gld<PS>(E + J0 + c);
        sm.put(c, p, (float)e);
    }
    // The slot key is the seed (0, cell 0) or a real pair of this sweep, so a
    // pair of ours can only win with delta < 0 (key delta 0) or delta <= key delta.
    // This tile's minimum of the previous sweep, if the move applied since leaves
    // it intact, is such a real pair too: it tightens the start bound and is
    // published for the other tiles.
    // kSweepLocal: the tile's own minimum over its improving pairs, independent
    // of every other tile (reused by the incremental sweep while the tile is clean)
    unsigned long long g = (flags & kSweepLocal) ? seed_key() : *(volatile unsigned long long*)&slot->key;
    if (!FIRST && !(flags & kSweepLocal) && (flags & kSweepSeed) && *(volatile int*)&slot->seed_ok) {
        const unsigned long long mv = *(volatile unsigned long long*)&slot->last_key;
        const unsigned long long k = surviving_key(*(volatile unsigned long long*)tilebest, key_i(mv), key_j(mv));
        if (k < g) {
            g = k;
            if (tid == 0) atomicMin(&slot->key, k);
        }
    }
    const int dg = key_delta(g);
    if (active) {
#pragma unroll
        for (int r = 0; r < R; r++) my_rowe[r] = erow[r];
    }
    if (WT) __syncwarp();
    else __syncthreads();

    unsigned long long mykey = kKeyNone;
    // FIRST: a tile whose lowest cell is above an improving pair already found
    // (the global key) cannot hold the first improving pair
    const bool skip = FIRST && g < pack_key(kFirstDelta, wrow0, jstart);
    if (active && !skip) {
        Bound<R> b;
        set_bound<R>(b, erow, FIRST ? 0 : (dg == 0 ? 0 : dg + 1));
        const bool masked = (wrow0 + 32 * R - 1) >= jstart;  // warp-uniform: some row >= some j
#ifdef TSP2OPT_TILE_TIMING
        const long long tt1 = clock64();
#endif
        if (!(flags & kSweepTileBounds) || tile_may_pass<R>(rows, b, sm, jstart - J0, J1 - J0)) {
#ifdef TSP2OPT_STATS
            if (lane == 0) atomicAdd(&g_stats[3], 1ULL);
#endif
            if (masked) walk<R, true, PS, FIRST>(rows, b, row0, jstart, J0, J1, sm, my_rowe, my_rowp, mykey, warp);
            else walk<R, false, PS, FIRST>(rows, b, row0, jstart, J0, J1, sm, my_rowe, my_rowp, mykey, warp);
#ifdef TSP2OPT_TILE_TIMING
            const long long tt2 = clock64();
            if (lane == 0) {
                atomicAdd(&g_stats[0], (unsigned long long)(tt1 - tt0));
                atomicAdd(&g_stats[1], (unsigned long long)(tt2 - tt1));
                atomicAdd(&g_stats[2], 1ULL);
                atomicMax(&g_stats[3], (unsigned long long)(tt2 - tt0));
            }
#endif
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            const unsigned long long other = __shfl_xor_sync(0xffffffffu, mykey, o);
            mykey = other < mykey ? other : mykey;
        }
        if (lane == 0 && mykey < *(volatile unsigned long long*)&slot->key) atomicMin(&slot->key, mykey);
    }
    // The tile's best (a real pair of this sweep, or none) is kept for the next
    // iteration's seed (apply_phase: moves the applied reversal leaves intact).
    if (WT) {
        if (lane == 0) *tilebest = active ? mykey : kKeyNone;  // mykey is the warp minimum here
        __syncwarp();
        return;
    }
    __shared__ unsigned long long s_red[kMaxWarpsPerTile];
    if (lane == 0) s_red[warp] = mykey;
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long m = s_red[0];
        for (int w = 1; w < (int)(blockDim.x >> 5); w++) m = s_red[w] < m ? s_red[w] : m;
        *tilebest = m;
    }
}

// One column part [jb, je) of a tile whose column chunk (from J0), row edges
// and row cities (rows [I0, I0 + 32 R]) a whole CTA has staged in `sm`, swept by
// ONE warp with the tile-local bound (kSweepLocal: delta < 0, the global key
// ignored), so the tile's minimum is the min over its parts and stays exact on
// its own.  The persistent incremental search splits each kept tile into parts
// over several warps (a warp alone on its SMSP walks a column step in about 500
// cycles of latency; the slowest whole-tile walk bounded the move).  The walk,
// the filters and the exact path are sweep_tile's; each part's column
// thresholds (slot 0 of the column records) are written only by the warp
// walking it.  Returns the lane's key (kKeyNone if none).
template <int R, bool FIRST>
__device__ __forceinline__ unsigned long long sweep_part(int I0, int J0, int jb, int je, const TileSmem& sm,
                                                         int flags)
{
    const int lane = threadIdx.x & 31;
    const int row0 = I0 + lane * R;
    const int jstart = max(jb, I0 + 1);  // no pair of the tile has j <= I0
    unsigned long long mykey = kKeyNone;
    if (jstart >= je) return mykey;  // warp-uniform
    const float* my_rowe = sm.rowe + lane * R;
    const float2* my_rowp = sm.rowp + lane * (R + 1);
    Rows<R> rows;
    float erow[R];
#pragma unroll
    for (int q = 0; q < (R + 1) / 2; q++) {
        const float2 p0 = my_rowp[2 * q], p1 = my_rowp[2 * q + 1];
        rows.xp[q] = make_float2(p0.x, p1.x);
        rows.yp[q] = make_float2(p0.y, p1.y);
    }
#pragma unroll
    for (int r = 0; r < R; r++) erow[r] = my_rowe[r];
    Bound<R> b;
    set_bound<R>(b, erow, 0);
    const bool masked = (I0 + 32 * R - 1) >= jstart;  // some row >= some column
    if (!(flags & kSweepPartBounds) || tile_may_pass<R>(rows, b, sm, jstart - J0, je - J0)) {
        if (masked) walk<R, true, true, FIRST>(rows, b, row0, jstart, J0, je, sm, my_rowe, my_rowp, mykey, 0);
        else walk<R, false, true, FIRST>(rows, b, row0, jstart, J0, je, sm, my_rowe, my_rowp, mykey, 0);
    }
    return mykey;
}

}  // namespace tsp2opt
