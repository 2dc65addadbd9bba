// tsp2opt_sweep25.cu -- best-improvement 2.5-opt (2-opt plus node insertion)
// on the device (L26 §VII "more complex local search
// algorithms such as 2.5-opt"; reading R19 in DESIGN.md §3).
//
// Neighbourhood: the pairs 0 <= i < j <= n-1 of the 2-opt sweep, three moves
// per pair (g_k = D(k-1, k+1) - e_{k-1} - e_k, the gain of removing city k):
//   type 0  2-opt:                          D(i,j) + D(i+1,j+1) - e_i - e_j
//   type 1  city i+1 into edge (j, j+1):    g_{i+1} + D(i+1,j) + D(i+1,j+1) - e_j   (j >= i+2)
//   type 2  city j into edge (i, i+1):      g_j + D(i,j) + D(i+1,j) - e_i           (j >= i+2)
// Best = lowest (delta, Fig. 3 cell, type) with delta < 0.  The sweep
// minimises the 2-opt key (delta, cell) over all three types -- the same key
// and reduction as the 2-opt sweep -- and the apply kernel resolves the type
// as the lowest one reaching that delta at that cell, which is the same
// order.
//
// The walk is the 2-opt walk of tsp2opt_sweep.cuh (R = 7 rows per lane,
// diagonal reuse): the lane already holds s(i_r, j) and s(i_r, j+1) for all
// its R+1 row cities, i.e. every distance the three moves need.  The exact
// necessary condition of DESIGN.md §5.2 extends per type with the same split
// a1 + a2 = B - 2 (delta <= B - 1 needs one of two halves to be small):
//   type 0:  D(i,j) <= e_i + a1        or  D(i+1,j+1) <= e_j + a2
//   type 1:  D(i+1,j) <= a1 - g_{i+1}  or  D(i+1,j+1) <= e_j + a2
//   type 2:  D(i,j) <= e_i + a1        or  D(i+1,j) <= a2 - g_j
// so per row city one merged threshold max(row-edge, row-gain) on s(i_r, j)
// (R+1 compares instead of R), the 2-opt column threshold on min_r s(i_r+1,
// j+1), and one more column threshold (a2 - g_j) on min_r s(i_r+1, j) -- the
// previous step's column minimum, carried in a register.
#include "tsp2opt_device.cuh"
#include "tsp2opt_internal.h"
#include "tsp2opt_sweep.cuh"

namespace tsp2opt {

namespace {

constexpr int R25 = kRowsSmall;  // 7 rows per lane: register room for the extra threshold

struct Tile25Smem {
    float4* colxy;  // [TJ + 2] (-x, -x, -y, -y) of columns J0.. and one spare
    float* cole;    // [TJ + 2] e_j
    float* colg;    // [TJ + 2] g_j
    float* rowe;    // [TI] e_i of the CTA's rows (lane stride R)
    float* rowg;    // [TI] g_{i+1} of the CTA's rows (lane stride R)
    __device__ Tile25Smem(void* base, int TJ, int TI)
        : colxy(reinterpret_cast<float4*>(base)),
          cole(reinterpret_cast<float*>(colxy + TJ + 2)),
          colg(cole + TJ + 2),
          rowe(colg + TJ + 2),
          rowg(rowe + TI)
    {
    }
};

struct Bound25 {
    int B;            // accept delta < B
    float Bf, a2f;
    float srow[R25 + 1];  // merged thresholds on s(i_k, j), k = 0..R
};

__device__ __forceinline__ void set_bound25(Bound25& b, const float* erow, const float* grow, int B)
{
    b.B = B;
    b.Bf = (float)B;
    const int c = B - 1;
    const int a1 = (c - 1) >> 1;
    const int a2 = c - 1 - a1;
    b.a2f = (float)a2;
    const float a1f = (float)a1;
#pragma unroll
    for (int k = 0; k <= R25; k++) {
        const float A = k < R25 ? sq_threshold(erow[k] + a1f) : -1.0f;    // type 0/2 of pair k
        const float F = k >= 1 ? sq_threshold(a1f - grow[k - 1]) : -1.0f;  // type 1 of pair k-1
        b.srow[k] = fmaxf(A, F);
    }
}

// exact nint distance of two biased points (float path when unambiguous)
__device__ __forceinline__ float edge25(float2 a, float bx_neg, float by_neg)
{
    const float dx = a.x + bx_neg, dy = a.y + by_neg;  // exact: biased floats share the exponent
    float d;
    if (nint_from_float(fmaf(dx, dx, dy * dy), d)) return d;
    return (float)exact_dist_xy(unbias(a.x), unbias(a.y), unbias(-bx_neg), unbias(-by_neg));
}

template <bool MASK, bool PS>
__device__ __forceinline__ void exact_step25(Bound25& b, const float (&cur)[R25 + 1], const float (&nxt)[R25 + 1],
                                             float scolB, float scolD, int row0, int j, float4 c0, float4 c1,
                                             float ej, float gj, const float* my_rowe, const float* my_rowg,
                                             const float2* P, unsigned long long& mykey)
{
    unsigned mask = 0;
#pragma unroll
    for (int r = 0; r < R25; r++) {
        bool cand = cur[r] <= b.srow[r] || nxt[r + 1] <= scolB || cur[r + 1] <= b.srow[r + 1] || cur[r + 1] <= scolD;
        if (MASK) cand = cand && (row0 + r < j);
        mask |= (cand ? 1u : 0u) << r;
    }
    float Bf = b.Bf;
    while (mask) {  // ascending r == ascending cell number
        const int r = __ffs(mask) - 1;
        mask &= mask - 1;
        const int i = row0 + r;
        const float2 pi = gld<PS>(P + i), pi1 = gld<PS>(P + i + 1);
        const float dij = edge25(pi, c0.x, c0.z), di1j1 = edge25(pi1, c1.x, c1.z);
        const float ei = my_rowe[r];
        float d = (dij + di1j1) - (ei + ej);  // exact: integers < 2^24
        if (j >= i + 2) {
            const float di1j = edge25(pi1, c0.x, c0.z);
            d = fminf(d, (my_rowg[r] + di1j) + (di1j1 - ej));  // type 1: city i+1 into (j, j+1)
            d = fminf(d, (gj + dij) + (di1j - ei));            // type 2: city j into (i, i+1)
        }
        if (d < Bf) {
            Bf = d;
            mykey = pack_key((int)d, i, j);
        }
    }
    if (Bf < b.Bf) {
        b.B = (int)Bf;
        b.Bf = Bf;
    }
}

template <bool MASK, bool PS>
__device__ __forceinline__ void column_step25(const Rows<R25>& rows, Bound25& b, const float (&cur)[R25 + 1],
                                              float (&nxt)[R25 + 1], float& mcur, int row0, int j, int J0,
                                              const Tile25Smem& sm, const float* my_rowe, const float* my_rowg,
                                              const float2* P, unsigned long long& mykey)
{
    const float4 c1 = sm.colxy[j + 1 - J0];
    column_sq<R25>(nxt, rows, c1);
    const float ej = sm.cole[j - J0], gj = sm.colg[j - J0];
    const float scolB = sq_threshold(ej + b.a2f);
    const float scolD = sq_threshold(b.a2f - gj);
    const float mnxt = tree_min<1, R25 + 1>(nxt);
    bool any;
    if (!MASK) {
        bool a0 = mnxt <= scolB, a1 = mcur <= scolD, a2 = false, a3 = false;
#pragma unroll
        for (int k = 0; k <= R25; k++) {
            const bool t = cur[k] <= b.srow[k];
            if ((k & 3) == 0) a0 |= t;
            else if ((k & 3) == 1) a1 |= t;
            else if ((k & 3) == 2) a2 |= t;
            else a3 |= t;
        }
        any = (a0 | a1) | (a2 | a3);
    } else {
        any = false;
#pragma unroll
        for (int r = 0; r < R25; r++)
            any |= (cur[r] <= b.srow[r] || nxt[r + 1] <= scolB || cur[r + 1] <= b.srow[r + 1] ||
                    cur[r + 1] <= scolD) &&
                   (row0 + r < j);
    }
    mcur = mnxt;
    if (__builtin_expect(__any_sync(0xffffffffu, any), 0)) {
        const int B0 = b.B;
        if (any)
            exact_step25<MASK, PS>(b, cur, nxt, scolB, scolD, row0, j, sm.colxy[j - J0], c1, ej, gj, my_rowe,
                                   my_rowg, P, mykey);
        const int wb = __reduce_min_sync(0xffffffffu, b.B);
        const int nb = min(b.B, wb + 1);
        if (nb < B0) set_bound25(b, my_rowe, my_rowg, nb);
    }
}

template <bool MASK, bool PS>
__device__ __forceinline__ void walk25(const Rows<R25>& rows, Bound25& b, int row0, int jstart, int J0, int J1,
                                       const Tile25Smem& sm, const float* my_rowe, const float* my_rowg,
                                       const float2* P, unsigned long long& mykey)
{
    float sa[R25 + 1], sb[R25 + 1];
    column_sq<R25>(sa, rows, sm.colxy[jstart - J0]);
    float mcur = tree_min<1, R25 + 1>(sa);
    int j = jstart;
    for (; j + 1 < J1; j += 2) {
        column_step25<MASK, PS>(rows, b, sa, sb, mcur, row0, j, J0, sm, my_rowe, my_rowg, P, mykey);
        column_step25<MASK, PS>(rows, b, sb, sa, mcur, row0, j + 1, J0, sm, my_rowe, my_rowg, P, mykey);
    }
    if (j < J1) column_step25<MASK, PS>(rows, b, sa, sb, mcur, row0, j, J0, sm, my_rowe, my_rowg, P, mykey);
}

// Tile-level form of the condition (as tile_may_pass of the 2-opt sweep): every
// squared distance the walk compares joins a city of the row block to a city
// of the column chunk, so it is >= the squared gap of the two boxes; every
// threshold is <= max(max_k srow[k], T(max e_j + a2), T(max(-g_j) + a2)).
__device__ __forceinline__ bool tile_may_pass25(const Rows<R25>& rows, const Bound25& b, const Tile25Smem& sm,
                                                int cbeg, int cend)
{
    float xlo = rows.xp[0].x, xhi = xlo, ylo = rows.yp[0].x, yhi = ylo;
#pragma unroll
    for (int q = 0; q < (R25 + 1) / 2; q++) {
        xlo = fminf(xlo, fminf(rows.xp[q].x, rows.xp[q].y));
        xhi = fmaxf(xhi, fmaxf(rows.xp[q].x, rows.xp[q].y));
        ylo = fminf(ylo, fminf(rows.yp[q].x, rows.yp[q].y));
        yhi = fmaxf(yhi, fmaxf(rows.yp[q].x, rows.yp[q].y));
    }
    float smax = b.srow[0];
#pragma unroll
    for (int k = 1; k <= R25; k++) smax = fmaxf(smax, b.srow[k]);
    float cxlo = 3.0e38f, cxhi = -3.0e38f, cylo = 3.0e38f, cyhi = -3.0e38f, emax = -1.0e30f, gneg = -1.0e30f;
    for (int c = cbeg + (int)(threadIdx.x & 31); c <= cend; c += 32) {
        const float4 v = sm.colxy[c];
        cxlo = fminf(cxlo, -v.x);
        cxhi = fmaxf(cxhi, -v.x);
        cylo = fminf(cylo, -v.z);
        cyhi = fmaxf(cyhi, -v.z);
        if (c < cend) {
            emax = fmaxf(emax, sm.cole[c]);
            gneg = fmaxf(gneg, -sm.colg[c]);
        }
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
        gneg = fmaxf(gneg, __shfl_xor_sync(0xffffffffu, gneg, o));
    }
    const float thr = fmaxf(smax, fmaxf(sq_threshold(emax + b.a2f), sq_threshold(gneg + b.a2f)));
    const float gx = fmaxf(0.f, fmaxf(cxlo - xhi, xlo - cxhi));
    const float gy = fmaxf(0.f, fmaxf(cylo - yhi, ylo - cyhi));
    const float d2 = fmaf(gx, gx, gy * gy);
    return d2 * 0.99999904632568359375f <= thr;  // (1 - 2^-20), as tile_may_pass
}

// exact g_k = D(k-1, k+1) - D(k-1, k) - D(k, k+1) of position k (closed tour)
__device__ __forceinline__ int gain_at(const float2* P, int n, int k)
{
    const int km = k == 0 ? n - 1 : k - 1;
    const float2 a = P[km], b = P[k], c = P[k + 1];
    return exact_dist_biased(a, c) - exact_dist_biased(a, b) - exact_dist_biased(b, c);
}

// the lowest move type reaching `delta` at (i, j) (the sweep's key carries no type)
__device__ __forceinline__ int move_type25(const float2* P, const int* E, const int* G, int i, int j, int delta)
{
    const float2 pi = P[i], pi1 = P[i + 1], pj = P[j], pj1 = P[j + 1];
    const int dij = exact_dist_biased(pi, pj), di1j1 = exact_dist_biased(pi1, pj1);
    if (dij + di1j1 - E[i] - E[j] == delta) return 0;
    if (j >= i + 2) {
        const int di1j = exact_dist_biased(pi1, pj);
        if (G[i + 1] + di1j + di1j1 - E[j] == delta) return 1;
        if (G[j] + dij + di1j - E[i] == delta) return 2;
    }
    return -1;
}

// delta of an explicit move (i, j, type) on the current state
__device__ __forceinline__ int move_delta25(const float2* P, const int* E, const int* G, int i, int j, int t)
{
    const float2 pi = P[i], pi1 = P[i + 1], pj = P[j], pj1 = P[j + 1];
    if (t == 0) return exact_dist_biased(pi, pj) + exact_dist_biased(pi1, pj1) - E[i] - E[j];
    const int di1j = exact_dist_biased(pi1, pj);
    if (t == 1) return G[i + 1] + di1j + exact_dist_biased(pi1, pj1) - E[j];
    return G[j] + exact_dist_biased(pi, pj) + di1j - E[i];
}

__device__ __forceinline__ void reverse_range(float2* P, int* tour, int lo, int hi, int gtid, int stride)
{
    const int half = (hi - lo + 1) >> 1;
    for (int t = gtid; t < half; t += stride) {
        const int a = lo + t, c = hi - t;
        const float2 pa = __ldcg(P + a), pc = __ldcg(P + c);
        P[a] = pc;
        P[c] = pa;
        const int ta = __ldcg(tour + a), tc = __ldcg(tour + c);
        tour[a] = tc;
        tour[c] = ta;
    }
}

}  // namespace

// a4 + a5 of the 2.5-opt sweep over one (row block x column chunk) tile.
// The caller synchronises the CTA before the shared chunk is reused.
__device__ __forceinline__ void sweep25_tile(const float2* __restrict__ P, const int* __restrict__ E,
                                             const int* __restrict__ G, int n, int2 tile, int TJ,
                                             Slot* __restrict__ slot, void* smem, int flags,
                                             unsigned long long* __restrict__ tilebest)
{
    const int TI = 32 * R25 * (int)(blockDim.x >> 5);
    const Tile25Smem sm(smem, TJ, TI);
    const int I0 = tile.x, J0 = tile.y;
    const int J1 = min(J0 + TJ, n);
    const int ncol = J1 - J0;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int wrow0 = I0 + warp * 32 * R25;
    const int row0 = wrow0 + lane * R25;
    const int jstart = max(J0, wrow0 + 1);
    const bool active = jstart < J1;
    float* my_rowe = sm.rowe + threadIdx.x * R25;
    float* my_rowg = sm.rowg + threadIdx.x * R25;

    Rows<R25> rows;
    float erow[R25], grow[R25];
    if (active) {
#pragma unroll
        for (int q = 0; q < (R25 + 1) / 2; q++) {
            const float2 p0 = __ldg(P + row0 + 2 * q), p1 = __ldg(P + row0 + 2 * q + 1);
            rows.xp[q] = make_float2(p0.x, p1.x);
            rows.yp[q] = make_float2(p0.y, p1.y);
        }
#pragma unroll
        for (int r = 0; r < R25; r++) {
            erow[r] = (float)__ldg(E + row0 + r);
            grow[r] = (float)__ldg(G + row0 + r + 1);
        }
    }
    for (int c = threadIdx.x; c <= ncol + 1; c += blockDim.x) {
        const float2 p = __ldg(P + J0 + c);
        sm.colxy[c] = make_float4(-p.x, -p.x, -p.y, -p.y);
        sm.cole[c] = (float)__ldg(E + J0 + c);
        sm.colg[c] = (float)__ldg(G + J0 + c);
    }
    // kSweepLocal: the tile's own minimum (reused by the incremental sweep while clean)
    const unsigned long long g = (flags & kSweepLocal) ? seed_key() : *(volatile unsigned long long*)&slot->key;
    const int dg = key_delta(g);
    if (active) {
#pragma unroll
        for (int r = 0; r < R25; r++) {
            my_rowe[r] = erow[r];
            my_rowg[r] = grow[r];
        }
    }
    __syncthreads();
    unsigned long long mykey = kKeyNone;
    if (active) {
        Bound25 b;
        set_bound25(b, erow, grow, dg == 0 ? 0 : dg + 1);
        const bool masked = (wrow0 + 32 * R25 - 1) >= jstart;
        if (!(flags & kSweepTileBounds) || tile_may_pass25(rows, b, sm, jstart - J0, J1 - J0)) {
            if (masked) walk25<true, false>(rows, b, row0, jstart, J0, J1, sm, my_rowe, my_rowg, P, mykey);
            else walk25<false, false>(rows, b, row0, jstart, J0, J1, sm, my_rowe, my_rowg, P, mykey);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            const unsigned long long other = __shfl_xor_sync(0xffffffffu, mykey, o);
            mykey = other < mykey ? other : mykey;
        }
        if (lane == 0 && mykey < *(volatile unsigned long long*)&slot->key) atomicMin(&slot->key, mykey);
    }
    if (tilebest) {  // the tile's minimum over its warps (incremental sweep)
        __shared__ unsigned long long s_red25[kMaxWarps];
        if (lane == 0) s_red25[warp] = mykey;
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned long long m = s_red25[0];
            for (int w = 1; w < (int)(blockDim.x >> 5); w++) m = s_red25[w] < m ? s_red25[w] : m;
            *tilebest = m;
        }
    }
}

__global__ void __launch_bounds__(128, 4) sweep25_kernel(const float2* __restrict__ P, const int* __restrict__ E,
                                                         const int* __restrict__ G, int n,
                                                         const int2* __restrict__ tiles, int TJ,
                                                         Slot* __restrict__ slot, int respect_done, int flags)
{
    extern __shared__ float4 smem25[];
    pdl_trigger();
    pdl_wait();
    if (respect_done && *(volatile int*)&slot->done) return;  // converged: iteration is a no-op
    sweep25_tile(P, E, G, n, tiles[blockIdx.x], TJ, slot, smem25, flags, nullptr);
}

// The 2.5-opt sweep over the culled list (as sweep_list_kernel: first entry
// static, then dynamic claims on slot->next_tile).
__global__ void __launch_bounds__(128, 4) sweep25_list_kernel(const float2* __restrict__ P,
                                                              const int* __restrict__ E, const int* __restrict__ G,
                                                              int n, const int4* __restrict__ list, int TJ,
                                                              Slot* __restrict__ slot, int respect_done,
                                                              unsigned long long* __restrict__ tilebest, int flags)
{
    extern __shared__ float4 smem25[];
    __shared__ int4 s_t;
    pdl_trigger();
    pdl_wait();
    const int done = respect_done ? *(volatile int*)&slot->done : 0;  // both fields in one round trip
    const unsigned count = *(volatile unsigned*)&slot->ncull;
    if (done) return;
    unsigned k = blockIdx.x;
    for (;;) {
        if (threadIdx.x == 0) s_t = k < count ? list[k] : make_int4(0, 0, -1, 0);
        __syncthreads();
        const int4 e = s_t;
        if (e.z < 0) break;
        sweep25_tile(P, E, G, n, make_int2(e.x, e.y), TJ, slot, smem25, flags | kSweepTileBounds,
                     (flags & kSweepIncremental) ? tilebest + e.z : nullptr);
        if (threadIdx.x == 0) k = gridDim.x + atomicAdd(&slot->next_tile, 1u);
        __syncthreads();
    }
}

// g_k for positions [lo, hi] (after a tour load / when the mode is switched on)
__global__ void gain_kernel(const float2* __restrict__ P, int* __restrict__ G, int n, int lo, int hi)
{
    for (int k = lo + blockIdx.x * blockDim.x + threadIdx.x; k <= hi; k += gridDim.x * blockDim.x)
        G[k] = gain_at(P, n, k);
}

// The type of the sweep's best key (tsp2opt_best_move_typed).
__global__ void decide25_kernel(const float2* __restrict__ P, const int* __restrict__ E, const int* __restrict__ G,
                                Slot* __restrict__ slot)
{
    const unsigned long long k = slot->key;
    slot->mtype = move_type25(P, E, G, key_i(k), key_j(k), key_delta(k));
}

// a7 + a8 for 2.5-opt (cooperative grid, grid barriers between phases):
// decide the move and its type from the pre-move state (every block reads
// before any block writes), reverse positions i+1..j, for a node insertion
// reverse i+1..j-1 (type 1: rotate left) or i+2..j (type 2: rotate right),
// then recompute the edges of positions i..j and the gains of i..j+1 (the only
// ones whose three cities moved).  Position 0 never moves, so P[n] = P[0]
// stays valid.
__global__ void __launch_bounds__(256) apply25_kernel(float2* __restrict__ P, int* __restrict__ E, int* __restrict__ G,
                                                      int* __restrict__ tour, int n, const Slot* __restrict__ in,
                                                      Slot* __restrict__ out, long long max_moves, int explicit_move,
                                                      int ei, int ej, int etype,
                                                      unsigned long long* __restrict__ trace, int* __restrict__ ttype,
                                                      long long trace_cap, unsigned* __restrict__ bar)
{
    __shared__ int s_i, s_j, s_t, s_apply;
    if (threadIdx.x == 0) {
        const unsigned long long key = *(volatile const unsigned long long*)&in->key;
        const int done = *(volatile const int*)&in->done;
        const long long moves = *(volatile const long long*)&in->moves;
        int i, j, t, delta;
        bool apply;
        if (explicit_move) {
            i = ei;
            j = ej;
            t = etype;
            delta = move_delta25(P, E, G, i, j, t);
            apply = true;
        } else {
            i = key_i(key);
            j = key_j(key);
            delta = key_delta(key);
            apply = !done && delta < 0 && moves < max_moves;
            t = apply ? move_type25(P, E, G, i, j, delta) : 0;
            if (t < 0) t = 0;  // cannot happen: the key's delta is one of the three
        }
        if (blockIdx.x == 0) {
            Slot o;
            o.key = seed_key();
            o.last_key = explicit_move ? in->last_key : key;
            o.moves = moves;
            o.length = in->length;
            o.done = explicit_move ? (done & 4) : done;
            o.next_tile = 0;
            o.ncull = 0;
            o.seed_ok = (apply && !explicit_move) ? 1 : 0;  // the incremental sweep may reuse clean tiles
            o.mtype = t;
            if (!explicit_move && !done) {
                if (delta >= 0) o.done = 1;              // local minimum (reading R7)
                else if (moves >= max_moves) o.done = 2;  // capped (reading R8)
            }
            if (apply) {
                o.length += delta;
                o.moves = moves + 1;
                if (trace && !explicit_move && moves < trace_cap) {
                    trace[moves] = key;
                    ttype[moves] = t;
                }
            }
            *out = o;
        }
        s_i = i;
        s_j = j;
        s_t = t;
        s_apply = apply ? 1 : 0;
    }
    __syncthreads();
    const int i = s_i, j = s_j, t = s_t;
    if (!s_apply) return;  // grid-uniform: every block decided the same
    const int gtid = blockIdx.x * blockDim.x + threadIdx.x, stride = gridDim.x * blockDim.x;
    grid_sync_gen(reinterpret_cast<unsigned long long*>(bar));  // all blocks have read the pre-move state
    reverse_range(P, tour, i + 1, j, gtid, stride);
    grid_sync_gen(reinterpret_cast<unsigned long long*>(bar));
    if (t == 1) reverse_range(P, tour, i + 1, j - 1, gtid, stride);
    else if (t == 2) reverse_range(P, tour, i + 2, j, gtid, stride);
    grid_sync_gen(reinterpret_cast<unsigned long long*>(bar));
    for (int k = i + gtid; k <= j; k += stride) E[k] = exact_dist_biased(__ldcg(P + k), __ldcg(P + k + 1));
    for (int x = i + gtid; x <= j + 1; x += stride) {
        const int k = x == n ? 0 : x;
        const int km = k == 0 ? n - 1 : k - 1;
        const float2 a = __ldcg(P + km), b = __ldcg(P + k), c = __ldcg(P + k + 1);
        G[k] = exact_dist_biased(a, c) - exact_dist_biased(a, b) - exact_dist_biased(b, c);
    }
}

// ---------------------------------------------------------------------------
size_t sweep25_smem_bytes(const Geometry& g)
{
    return (size_t)(g.tj + 2) * (sizeof(float4) + 2 * sizeof(float)) + (size_t)2 * g.ti() * sizeof(float);
}

cudaError_t sweep25_prepare()
{
    const int bytes = (int)sweep25_smem_bytes(Geometry{R25, kMaxWarps, kMaxTJ});
    cudaError_t e = cudaFuncSetAttribute(sweep25_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e != cudaSuccess) return e;
    return cudaFuncSetAttribute(sweep25_list_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
}

int sweep25_list_grid(const Geometry& g, int ntiles)
{
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, sweep25_list_kernel, 32 * g.warps,
                                                      sweep25_smem_bytes(g)) != cudaSuccess)
        return 0;
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    return std::min(per_sm * sms, ntiles);
}

cudaError_t launch_sweep25_list(const Geometry& g, const float2* P, const int* E, const int* G, int n,
                                const int4* list, int grid, Slot* slot, int respect_done,
                                unsigned long long* tilebest, int flags, cudaStream_t st)
{
    if (flags & kSweepIncremental) flags = (flags | kSweepLocal) & ~kSweepSeed;
    if (grid <= 0) return cudaSuccess;
    if (g.rows != R25) return cudaErrorInvalidValue;
    cudaError_t e = launch_kernel_pdl(sweep25_list_kernel, dim3(grid), dim3(32 * g.warps), sweep25_smem_bytes(g), st,
                                      P, E, G, n, list, g.tj, slot, respect_done, tilebest, flags);
    if (e != cudaSuccess) return e;
    count_launch(1);
    return cudaGetLastError();
}

cudaError_t launch_sweep25(const Geometry& g, const float2* P, const int* E, const int* G, int n, const int2* tiles,
                           int ntiles, Slot* slot, int respect_done, int flags, cudaStream_t st)
{
    if (ntiles <= 0) return cudaSuccess;
    if (g.rows != R25) return cudaErrorInvalidValue;
    cudaError_t e = launch_kernel_pdl(sweep25_kernel, dim3(ntiles), dim3(32 * g.warps), sweep25_smem_bytes(g), st, P,
                                      E, G, n, tiles, g.tj, slot, respect_done, flags);
    if (e != cudaSuccess) return e;
    count_launch(1);
    return cudaGetLastError();
}

cudaError_t launch_gain(const float2* P, int* G, int n, int lo, int hi, cudaStream_t st)
{
    const int work = hi - lo + 1;
    gain_kernel<<<std::max(1, std::min(4 * 148, (work + 255) / 256)), 256, 0, st>>>(P, G, n, lo, hi);
    count_launch(1);
    return cudaGetLastError();
}

cudaError_t launch_decide25(const float2* P, const int* E, const int* G, Slot* slot, cudaStream_t st)
{
    decide25_kernel<<<1, 1, 0, st>>>(P, E, G, slot);
    count_launch(1);
    return cudaGetLastError();
}

cudaError_t launch_apply25(float2* P, int* E, int* G, int* tour, int n, const Slot* in, Slot* out,
                           long long max_moves, int explicit_move, int ei, int ej, int etype,
                           unsigned long long* trace, int* ttype, long long trace_cap, unsigned* bar, cudaStream_t st)
{
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int grid = std::max(1, std::min(sms, (n / 2 + 255) / 256));
    void* args[] = {&P, &E, &G, &tour, &n, &in, &out, &max_moves, &explicit_move, &ei, &ej, &etype, &trace, &ttype,
                    &trace_cap, &bar};
    count_launch(1);
    return cudaLaunchCooperativeKernel((const void*)apply25_kernel, dim3(grid), dim3(256), args, 0, st);
}

}  // namespace tsp2opt
