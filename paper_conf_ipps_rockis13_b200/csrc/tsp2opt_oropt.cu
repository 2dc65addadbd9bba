// tsp2opt_oropt.cu -- Or-opt sweep and apply (SURVEY.md §8(f) NEXT-4,
// "2.5-opt/Or-opt variants"; L26 §VII; reading R21 and §5.15).
//
// Neighbourhood (reading R21): the pairs 0 <= i < j <= n-1 of the closed tour
// (reading R1), 13 moves per pair: type 0 the 2-opt move, and for
// type = 1 + 4(L-1) + 2 dir + rev with j >= i+L+1 the move of a segment of
// L = 1..3 cities (dir 0: t[i+1..i+L] into the edge (t_j, t_{j+1}); dir 1:
// t[j-L+1..j] into the edge (t_i, t_{i+1})), reversed iff rev.  Best = the
// lowest (delta, Fig. 3 cell, type) with delta < 0, else (0, 1, type 0).
//
// Layout: Q[p] = coords[tour[p]] for p < n + 5 (positions mod n: the closed
// array of reading R10 plus the halo a segment of three past position n-1
// can reach), int2, and per-position removal-gain constants CR / CC.  The
// sweep (or_tile_kernel) walks (row block x column chunk)
// tiles, one row city per thread, with a 4 x 4 register window of distances
// sliding along the columns; from n > 2048 the window is FP32 with an exact
// fallback.  The packed key (delta + 2^18) << 44 | j << 24 | i << 4 | type
// (n <= 2^20) reduces per warp by shuffles, per CTA in shared memory and per
// GPU with one 64-bit atomicMin.  Exact distances are the EUC_2D nint of
// tsp2opt_device.cuh.  The apply writes positions i+1..j in their new order
// into a scratch span, then copies it back (two launches, no grid barrier).
// or_sweep_kernel (one thread per cell) is the first version, kept behind
// TSP2OPT_OROPT_NAIVE=1.
#include <atomic>
#include <climits>
#include <cstdlib>

#include "tsp2opt_internal.h"

namespace tsp2opt {

constexpr int kOrHalo = 5;
constexpr int kOrThreads = 256;

__host__ __device__ __forceinline__ unsigned long long or_pack(int delta, int i, int j, int type)
{
    return ((unsigned long long)(delta + kDeltaBias) << 44) | ((unsigned long long)j << 24) |
           ((unsigned long long)i << 4) | (unsigned long long)type;
}

__device__ __forceinline__ int or_d(int2 a, int2 b) { return exact_dist_xy(a.x, a.y, b.x, b.y); }

// Q[p] = coords[tour[p mod n]] for p < n + kOrHalo
__global__ void or_gather_kernel(const int* __restrict__ coords, const int* __restrict__ tour, int2* __restrict__ Q,
                                 int n)
{
    for (int p = blockIdx.x * blockDim.x + threadIdx.x; p < n + kOrHalo; p += gridDim.x * blockDim.x) {
        const int c = tour[p % n];
        Q[p] = make_int2(coords[2 * c], coords[2 * c + 1]);
    }
}

// Tour length: sum of d(Q[p], Q[p+1]), p < n, into *len (zeroed by the caller)
__global__ void or_length_kernel(const int2* __restrict__ Q, int n, unsigned long long* len)
{
    unsigned long long s = 0;
    for (int p = blockIdx.x * blockDim.x + threadIdx.x; p < n; p += gridDim.x * blockDim.x) s += or_d(Q[p], Q[p + 1]);
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if ((threadIdx.x & 31) == 0 && s) atomicAdd(len, s);
}

__global__ void __launch_bounds__(kOrThreads) or_sweep_kernel(const int2* __restrict__ Q, int n, long long cells,
                                                              unsigned long long* slot)
{
    if (*(volatile const unsigned long long*)(slot + kOrDone)) return;
    unsigned long long best = or_pack(0, 0, 1, 0);
    for (long long k = blockIdx.x * (long long)blockDim.x + threadIdx.x; k < cells;
         k += (long long)gridDim.x * blockDim.x) {
        // cell k = j(j-1)/2 + i (Fig. 3): j = floor((1 + sqrt(1 + 8k)) / 2), fixed up exactly
        int j = (int)((1.0 + sqrt(1.0 + 8.0 * (double)k)) * 0.5);
        while ((long long)j * (j - 1) / 2 > k) j--;
        while ((long long)(j + 1) * j / 2 <= k) j++;
        const int i = (int)(k - (long long)j * (j - 1) / 2);
        const int2 a0 = Q[i], a1 = Q[i + 1], bj = Q[j], bj1 = Q[j + 1];
        const int ei = or_d(a0, a1), ej = or_d(bj, bj1);
        int d = or_d(a0, bj) + or_d(a1, bj1) - ei - ej;  // type 0
        unsigned long long key = or_pack(d, i, j, 0);
        if (key < best) best = key;
#pragma unroll
        for (int L = 1; L <= 3; L++) {
            if (j < i + L + 1) break;
            // forward: t[i+1..i+L] into (t_j, t_{j+1})
            const int2 s0 = Q[i + 1], sL = Q[i + L], nx = Q[i + L + 1];
            const int rem_f = or_d(a0, nx) - ei - or_d(sL, nx) - ej;
            // backward: t[j-L+1..j] into (t_i, t_{i+1})
            const int2 pv = Q[j - L], u0 = Q[j - L + 1];
            const int rem_b = or_d(pv, bj1) - or_d(pv, u0) - ej - ei;
            const int df0 = rem_f + or_d(bj, s0) + or_d(sL, bj1);
            const int df1 = rem_f + or_d(bj, sL) + or_d(s0, bj1);
            const int db0 = rem_b + or_d(a0, u0) + or_d(bj, a1);
            const int db1 = rem_b + or_d(a0, bj) + or_d(u0, a1);
            const int t0 = 1 + 4 * (L - 1);
            key = or_pack(df0, i, j, t0);
            if (key < best) best = key;
            key = or_pack(df1, i, j, t0 + 1);
            if (key < best) best = key;
            key = or_pack(db0, i, j, t0 + 2);
            if (key < best) best = key;
            key = or_pack(db1, i, j, t0 + 3);
            if (key < best) best = key;
        }
    }
    for (int o = 16; o; o >>= 1) {
        const unsigned long long other = __shfl_xor_sync(0xffffffffu, best, o);
        best = other < best ? other : best;
    }
    __shared__ unsigned long long red[kOrThreads / 32];
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = best;
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 1; w < kOrThreads / 32; w++) best = red[w] < best ? red[w] : best;
        atomicMin(slot, best);
    }
}

// Per-position constants of the tiled sweep, rebuilt before every sweep (O(n)):
//   CR[p] = (e_p, rf_1, rf_2, rf_3) with rf_L = d(t_p, t_{p+L+1}) - e_p - d(t_{p+L}, t_{p+L+1})
//           (the row part of a forward move's removal gain);
//   CC[p] = (e_p, rb_1, rb_2, rb_3) with rb_L = d(t_{p-L}, t_{p+1}) - d(t_{p-L}, t_{p-L+1}) - e_p
//           (the column part of a backward move's removal gain; p - L >= 0 only is ever read).
__global__ void or_consts_kernel(const int2* __restrict__ Q, int n, int4* __restrict__ CR, int4* __restrict__ CC,
                                 unsigned long long* slot)
{
    if (*(volatile const unsigned long long*)(slot + kOrDone)) return;  // converged / capped: a no-op iteration
    if (blockIdx.x == 0 && threadIdx.x == 0) *slot = or_pack(0, 0, 1, 0);  // the sweep's seed key (reading R7)
    for (int p = blockIdx.x * blockDim.x + threadIdx.x; p < n; p += gridDim.x * blockDim.x) {
        const int e = or_d(Q[p], Q[p + 1]);
        int rf[3], rb[3];
#pragma unroll
        for (int L = 1; L <= 3; L++) {
            rf[L - 1] = or_d(Q[p], Q[p + L + 1]) - e - or_d(Q[p + L], Q[p + L + 1]);
            rb[L - 1] = p - L >= 0 ? or_d(Q[p - L], Q[p + 1]) - or_d(Q[p - L], Q[p - L + 1]) - e : 0;
        }
        CR[p] = make_int4(e, rf[0], rf[1], rf[2]);
        CC[p] = make_int4(e, rb[0], rb[1], rb[2]);
    }
}

constexpr int kOrMaxTI = 256;  // rows per tile = threads per CTA (one row city per thread), upper bound

// Tile geometry by size: enough CTAs to fill 148 SMs at small n, long column
// walks (few window warm-ups) at large n.
static void or_tiles(int n, int* ti, int* tj)
{
    if (n <= 2048) { *ti = 64; *tj = 16; }
    else if (n <= 16384) { *ti = 128; *tj = 32; }
    else { *ti = 256; *tj = 128; }
}

// The 13 moves of pair (i, j) from the window D_r[k] = d(t_{i+r}, t_{j-2+k})
// (columns j-2, j-1, j, j+1) and the per-position constants: min over the
// valid types of delta * 16 + type.
//   forward L:  rf_L - e_j + d(t_j, a) + d(b, t_{j+1}); a, b = t_{i+1}, t_{i+L} (rev: swapped)
//   backward L: rb_L - e_i + d(t_i, a) + d(b, t_{i+1}); a, b = t_{j-L+1}, t_j (rev: swapped)
// (moves of length L need gap = j - i >= L + 1; the L = 1 reversed types
// duplicate types 1 and 3 and never win the type tie-break.)
__device__ __forceinline__ int or_eval_exact(const int* D0, const int* D1, const int* D2, const int* D3, int4 cr,
                                             int4 cc, int gap)
{
    int v = (D0[2] + D1[3] - cr.x - cc.x) * 16;  // type 0
    if (gap >= 2) {
        const int f = cr.y - cc.x, b = cc.y - cr.x;
        v = min(v, (f + D1[2] + D1[3]) * 16 + 1);
        v = min(v, (b + D0[2] + D1[2]) * 16 + 3);
    }
    if (gap >= 3) {
        const int f = cr.z - cc.x, b = cc.z - cr.x;
        v = min(v, (f + D1[2] + D2[3]) * 16 + 5);
        v = min(v, (f + D2[2] + D1[3]) * 16 + 6);
        v = min(v, (b + D0[1] + D1[2]) * 16 + 7);
        v = min(v, (b + D0[2] + D1[1]) * 16 + 8);
    }
    if (gap >= 4) {
        const int f = cr.w - cc.x, b = cc.w - cr.x;
        v = min(v, (f + D1[2] + D3[3]) * 16 + 9);
        v = min(v, (f + D3[2] + D1[3]) * 16 + 10);
        v = min(v, (b + D0[0] + D1[2]) * 16 + 11);
        v = min(v, (b + D0[2] + D1[0]) * 16 + 12);
    }
    return v;
}

// The same minimum over the types in FP32 from approximate distances
// sqrt_approx(s_f), without the type.  Each distance is within 0.53 of its
// nint (0.5 rounding + 0.03 MUFU / s_f error, tsp2opt_selftest_sqrt), a move
// has two varying distances, and the three FP32 additions of values below
// 2^18 round by at most 0.05, so every exact delta is >= this value - 1.11.
__device__ __forceinline__ float or_eval_float(const float* F0, const float* F1, const float* F2, const float* F3,
                                               int4 cr, int4 cc, int gap)
{
    float m = F0[2] + F1[3] + (float)(-cr.x - cc.x);
    if (gap >= 2) {
        const float f = (float)(cr.y - cc.x), b = (float)(cc.y - cr.x);
        m = fminf(m, fminf(f + (F1[2] + F1[3]), b + (F0[2] + F1[2])));
    }
    if (gap >= 3) {
        const float f = (float)(cr.z - cc.x), b = (float)(cc.z - cr.x);
        m = fminf(m, fminf(f + fminf(F1[2] + F2[3], F2[2] + F1[3]), b + fminf(F0[1] + F1[2], F0[2] + F1[1])));
    }
    if (gap >= 4) {
        const float f = (float)(cr.w - cc.x), b = (float)(cc.w - cr.x);
        m = fminf(m, fminf(f + fminf(F1[2] + F3[3], F3[2] + F1[3]), b + fminf(F0[0] + F1[2], F0[2] + F1[0])));
    }
    return m;
}

constexpr float kOrSlack = 1.25f;  // > 1.11: a pair can beat `best` only if its float minimum <= best - 1 + kOrSlack

__device__ __forceinline__ float or_df(float2 a, float2 b)
{
    const float dx = a.x - b.x, dy = a.y - b.y;
    return sqrt_approx(fmaf(dx, dx, dy * dy));
}

// Tiled sweep: CTA = one (row block blockIdx.y, column chunk blockIdx.x) tile,
// thread = row i, walking the tile's columns j in increasing order.  Every
// distance of a pair's 13 moves is d(t_{i+r}, t_c) for r in 0..3 and c in
// j-2..j+1 (or a per-position constant), so a 4 x 4 register window slides
// along j and each column step computes only the 4 distances to t_{j+1}.
// The thread keeps its lowest (delta, cell, type): per pair the min of
// delta << 4 | type (lowest type among equal deltas), replacing the thread's
// best only on a strictly lower delta (cells increase along the walk).
// FILTER: the window holds FP32 approximate distances; a pair is evaluated
// exactly (12 exact distances from the coordinates) only when its FP32
// minimum can beat the thread's best (or_eval_float's bound).
template <bool FILTER>
__global__ void __launch_bounds__(kOrMaxTI) or_tile_kernel(const int2* __restrict__ Q, const int4* __restrict__ CR,
                                                           const int4* __restrict__ CC, int n, int tj,
                                                           unsigned long long* slot)
{
    const int ti = blockDim.x;
    const int row0 = blockIdx.y * ti, col1 = (blockIdx.x + 1) * tj;
    if (col1 - 1 <= row0) return;  // below the diagonal: no pair i < j (uniform over the CTA)
    if (*(volatile const unsigned long long*)(slot + kOrDone)) return;  // converged / capped
    const int i = row0 + threadIdx.x;
    const int j0 = max(blockIdx.x * tj, i + 1), j1 = min(n, col1);
    // Seed the thread's bound with the sweep's best so far (other CTAs'
    // atomicMin): only pairs with delta <= that delta can still win, and an
    // equal delta may win on a lower cell, so the bound is one above it.
    const int gd = (int)(*(volatile const unsigned long long*)slot >> 44) - kDeltaBias;
    int best = gd < 0 ? gd + 1 : 0, bj = 0, bt = 0;  // record a pair iff its delta < best; its column and type
    if (FILTER && i < n - 1 && j0 < j1) {
        const int2 r0 = Q[i], r1 = Q[i + 1], r2 = Q[i + 2], r3 = Q[i + 3];
        const float2 g0 = make_float2(r0.x, r0.y), g1 = make_float2(r1.x, r1.y), g2 = make_float2(r2.x, r2.y),
                     g3 = make_float2(r3.x, r3.y);
        const int4 cr = CR[i];
        float F0[4], F1[4], F2[4], F3[4];
#pragma unroll
        for (int k = 0; k < 3; k++) {
            const int2 q = Q[max(0, j0 - 2 + k)];
            const float2 c = make_float2(q.x, q.y);
            F0[k + 1] = or_df(g0, c);
            F1[k + 1] = or_df(g1, c);
            F2[k + 1] = or_df(g2, c);
            F3[k + 1] = or_df(g3, c);
        }
        for (int j = j0; j < j1; j++) {
#pragma unroll
            for (int k = 0; k < 3; k++) {
                F0[k] = F0[k + 1];
                F1[k] = F1[k + 1];
                F2[k] = F2[k + 1];
                F3[k] = F3[k + 1];
            }
            const int2 q = Q[j + 1];
            const float2 c = make_float2(q.x, q.y);
            F0[3] = or_df(g0, c);
            F1[3] = or_df(g1, c);
            F2[3] = or_df(g2, c);
            F3[3] = or_df(g3, c);
            const int4 cc = CC[j];
            const int gap = j - i;
            if (or_eval_float(F0, F1, F2, F3, cr, cc, gap) <= (float)(best - 1) + kOrSlack) {
                int D0[4], D1[4], D2[4], D3[4];
#pragma unroll
                for (int k = 0; k < 4; k++) {
                    const int2 w = Q[max(0, j - 2 + k)];
                    D0[k] = or_d(r0, w);
                    D1[k] = or_d(r1, w);
                    D2[k] = or_d(r2, w);
                    D3[k] = or_d(r3, w);
                }
                const int v = or_eval_exact(D0, D1, D2, D3, cr, cc, gap);
                if ((v >> 4) < best) {
                    best = v >> 4;
                    bt = v & 15;
                    bj = j;
                }
            }
        }
    }
    if (!FILTER && i < n - 1 && j0 < j1) {
        const int2 r0 = Q[i], r1 = Q[i + 1], r2 = Q[i + 2], r3 = Q[i + 3];
        const int4 cr = CR[i];
        // window D[r][k]: d(t_{i+r}, t_{j-2+k}), k = 0..3 (columns j-2, j-1, j, j+1); columns < 0 are never read
        int D0[4], D1[4], D2[4], D3[4];
#pragma unroll
        for (int k = 0; k < 3; k++) {
            const int2 c = Q[max(0, j0 - 2 + k)];
            D0[k + 1] = or_d(r0, c);
            D1[k + 1] = or_d(r1, c);
            D2[k + 1] = or_d(r2, c);
            D3[k + 1] = or_d(r3, c);
        }
        for (int j = j0; j < j1; j++) {
#pragma unroll
            for (int k = 0; k < 3; k++) {
                D0[k] = D0[k + 1];
                D1[k] = D1[k + 1];
                D2[k] = D2[k + 1];
                D3[k] = D3[k + 1];
            }
            const int2 c = Q[j + 1];
            D0[3] = or_d(r0, c);
            D1[3] = or_d(r1, c);
            D2[3] = or_d(r2, c);
            D3[3] = or_d(r3, c);
            const int v = or_eval_exact(D0, D1, D2, D3, CR[i], CC[j], j - i);
            if ((v >> 4) < best) {
                best = v >> 4;
                bt = v & 15;
                bj = j;
            }
        }
    }
    unsigned long long key = bj > 0 ? or_pack(best, i, bj, bt) : or_pack(0, 0, 1, 0);
    for (int o = 16; o; o >>= 1) {
        const unsigned long long other = __shfl_xor_sync(0xffffffffu, key, o);
        key = other < key ? other : key;
    }
    __shared__ unsigned long long red[kOrMaxTI / 32];
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = key;
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 1; w < (int)(blockDim.x >> 5); w++) key = red[w] < key ? red[w] : key;
        if (key < or_pack(0, 0, 1, 0)) atomicMin(slot, key);
    }
}

// span[p - i - 1] = the tour city that lands on position p in [i+1, j] (oracleor_apply's order)
// The move decision of one iteration, on the device (one thread): the sweep's
// key in slot[0]; slot[kOrDone] = 1 at a local minimum (delta >= 0, reading
// R7), 2 when capped with an improving move left (R8); otherwise the move is
// recorded (length, moves, trace row (i, j, delta, type)) and published in
// slot[kOrMove] for the apply kernels (0: no move this iteration).
__global__ void or_decide_kernel(unsigned long long* slot, int* __restrict__ trace, long long trace_cap)
{
    if (slot[kOrDone]) return;
    const unsigned long long key = slot[0];
    const int d = (int)(key >> 44) - kDeltaBias;
    const long long moves = (long long)slot[kOrMoves];
    if (d >= 0) {
        slot[kOrDone] = 1;
        slot[kOrMove] = 0;
        return;
    }
    if (moves >= (long long)slot[kOrCap]) {
        slot[kOrDone] = 2;
        slot[kOrMove] = 0;
        return;
    }
    const int j = (int)((key >> 24) & 0xFFFFF), i = (int)((key >> 4) & 0xFFFFF), type = (int)(key & 0xF);
    if (trace && moves < trace_cap) {
        trace[4 * moves] = i;
        trace[4 * moves + 1] = j;
        trace[4 * moves + 2] = d;
        trace[4 * moves + 3] = type;
    }
    slot[kOrLength] = (unsigned long long)((long long)slot[kOrLength] + d);
    slot[kOrMoves] = (unsigned long long)(moves + 1);
    slot[kOrMove] = key;
}

// span[p - i - 1] = the tour city that lands on position p in [i+1, j] (oracleor_apply's order),
// for the move the decide kernel published (none: a no-op)
__global__ void or_span_kernel(const int* __restrict__ tour, int* __restrict__ span,
                               const unsigned long long* __restrict__ slot)
{
    const unsigned long long key = slot[kOrMove];
    if (!key) return;
    const int j = (int)((key >> 24) & 0xFFFFF), i = (int)((key >> 4) & 0xFFFFF), type = (int)(key & 0xF);
    const int m = j - i;
    const int L = 1 + (type - 1) / 4, dir = ((type - 1) / 2) & 1, rev = (type - 1) & 1;
    for (int q = blockIdx.x * blockDim.x + threadIdx.x; q < m; q += gridDim.x * blockDim.x) {
        const int p = i + 1 + q;
        int src;
        if (type == 0) src = i + 1 + j - p;
        else if (dir == 0) src = p <= j - L ? p + L : (rev ? i + L - (p - (j - L + 1)) : i + 1 + (p - (j - L + 1)));
        else src = p <= i + L ? (rev ? j - (p - i - 1) : j - L + 1 + (p - i - 1)) : p - L;
        span[q] = tour[src];
    }
}

__global__ void or_commit_kernel(const int* __restrict__ coords, const int* __restrict__ span, int* __restrict__ tour,
                                 int2* __restrict__ Q, int n, const unsigned long long* __restrict__ slot)
{
    const unsigned long long key = slot[kOrMove];
    if (!key) return;
    const int j = (int)((key >> 24) & 0xFFFFF), i = (int)((key >> 4) & 0xFFFFF);
    for (int q = blockIdx.x * blockDim.x + threadIdx.x; q < j - i; q += gridDim.x * blockDim.x) {
        const int p = i + 1 + q, c = span[q];
        tour[p] = c;
        const int2 v = make_int2(coords[2 * c], coords[2 * c + 1]);
        Q[p] = v;
        if (p < kOrHalo) Q[n + p] = v;  // the halo copies of positions 1..4
    }
}

__global__ void or_seed_kernel(unsigned long long* slot)
{
    if (!slot[kOrDone]) slot[0] = or_pack(0, 0, 1, 0);
}

static int or_grid(long long work, int per_cta, int cap)
{
    int sms = 148;
    int dev = 0;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const long long need = (work + per_cta - 1) / per_cta;
    const long long g = std::min<long long>(need, (long long)sms * cap);
    return (int)std::max<long long>(1, g);
}

size_t oropt_q_entries(int n) { return (size_t)n + kOrHalo; }

cudaError_t launch_or_load(const int* coords, const int* tour, int2* Q, int n, unsigned long long* len, cudaStream_t st)
{
    cudaError_t e = cudaMemsetAsync(len, 0, sizeof(unsigned long long), st);
    if (e != cudaSuccess) return e;
    or_gather_kernel<<<or_grid(n + kOrHalo, 256, 4), 256, 0, st>>>(coords, tour, Q, n);
    or_length_kernel<<<or_grid(n, 256, 4), 256, 0, st>>>(Q, n, len);
    count_launch(2);
    return cudaGetLastError();
}

// Kernel and filter selection of the Or-opt sweep (none changes a result).
// Defaults come from TSP2OPT_OROPT_NAIVE / TSP2OPT_OROPT_FILTER, read once;
// tsp2opt_oropt_config overrides them (tests run every mode in one process).
// The FP32 filter pays from the 128 x 32 tiles up (measured: C3 / C4 sweeps
// 1.3x / 1.6x faster); the 16-column walks of n <= 2048 re-seed too often.
static std::atomic<int> g_or_filter{-2};  // -2 unset, -1 auto (n > 2048), 0 off, 1 on
static std::atomic<int> g_or_naive{-1};   // -1 unset, 0 tiled kernel, 1 one thread per cell

static bool or_naive()
{
    int v = g_or_naive.load();
    if (v < 0) {
        const char* s = getenv("TSP2OPT_OROPT_NAIVE");
        v = (s && s[0] == '1') ? 1 : 0;
        g_or_naive.store(v);
    }
    return v == 1;
}

static bool or_filter(int n)
{
    int m = g_or_filter.load();
    if (m == -2) {
        const char* s = getenv("TSP2OPT_OROPT_FILTER");
        m = s && (s[0] == '0' || s[0] == '1') ? s[0] - '0' : -1;
        g_or_filter.store(m);
    }
    return m < 0 ? n > 2048 : m == 1;
}

void or_config(int filter, int naive)
{
    g_or_filter.store(filter);
    g_or_naive.store(naive);
}

size_t oropt_const_entries(int n) { return (size_t)n; }

cudaError_t launch_or_sweep(const int2* Q, int4* CR, int4* CC, int n, unsigned long long* slot, cudaStream_t st)
{
    if (or_naive()) {  // TSP2OPT_OROPT_NAIVE=1: the one-thread-per-cell kernel (experiment switch, same result)
        or_seed_kernel<<<1, 1, 0, st>>>(slot);
        const long long cells = (long long)n * (n - 1) / 2;
        or_sweep_kernel<<<or_grid(cells, kOrThreads, 8), kOrThreads, 0, st>>>(Q, n, cells, slot);
        count_launch();
        return cudaGetLastError();
    }
    or_consts_kernel<<<or_grid(n, 256, 4), 256, 0, st>>>(Q, n, CR, CC, slot);  // also writes the seed key
    int ti, tj;
    or_tiles(n, &ti, &tj);
    const dim3 grid((n + tj - 1) / tj, (n + ti - 1) / ti);
    if (or_filter(n))
        or_tile_kernel<true><<<grid, ti, 0, st>>>(Q, CR, CC, n, tj, slot);
    else
        or_tile_kernel<false><<<grid, ti, 0, st>>>(Q, CR, CC, n, tj, slot);
    count_launch(2);
    return cudaGetLastError();
}

cudaError_t launch_or_apply(const int* coords, int* tour, int2* Q, int* span, int n, unsigned long long* slot,
                            int* trace, long long trace_cap, cudaStream_t st)
{
    const int g = or_grid(n, 256, 4);
    or_decide_kernel<<<1, 1, 0, st>>>(slot, trace, trace_cap);
    or_span_kernel<<<g, 256, 0, st>>>(tour, span, slot);
    or_commit_kernel<<<g, 256, 0, st>>>(coords, span, tour, Q, n, slot);
    count_launch(3);
    return cudaGetLastError();
}

void or_unpack(unsigned long long key, int* i, int* j, int* type, int* delta)
{
    *delta = (int)(key >> 44) - kDeltaBias;
    *j = (int)((key >> 24) & 0xFFFFF);
    *i = (int)((key >> 4) & 0xFFFFF);
    *type = (int)(key & 0xF);
}

}  // namespace tsp2opt
