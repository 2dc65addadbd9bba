// tsp2opt_sweep_xf.cuh -- "expanded form" fast path of the tile sweep.
//
// Same tile, lanes, reuse and exactness contract as tsp2opt_sweep.cuh (read
// that header first); only the fast per-pair filter is computed differently.
// With per-tile centred coordinates p' = p - c (c = a city of the tile) the
// squared distance of row r to column k is
//     s(r,k) = Q_r + Q_k - 2 p'_r . p'_k ,   Q = |p'|^2,
// so   u_r(k) := Q_r - 2 p'_r . p'_k = s(r,k) - Q_k
// costs two FFMA2 per PAIR of rows (vs FADD2, FADD2, FMUL2, FFMA2 for the
// direct dx^2 + dy^2), and both tests of DESIGN.md §5.2 become comparisons of
// minima against one value per column:
//   row test   s(r,j)     <= S_r  <=>  u_r(j) - S_r  <= -Q_j     (min over r)
//   col test   s(r+1,j+1) <= S_j  <=>  u_r(j+1)      <= S_j - Q_{j+1}
// The float error of u is bounded RELATIVE to Q_r + Q_k (each rounding is at
// most 2^-24 of a magnitude <= 2 (Q_r + Q_k) by 2|a||b| <= |a|^2 + |b|^2), so
// the thresholds carry separable margins -- 2^-18 of S and Q on the row side,
// 2^-18 of Q on the column side, plus 1 -- that dominate every rounding (proof
// in DESIGN.md §5.2b).  The filter therefore still never rejects a pair the
// exact test accepts; pairs that pass go through the same rare path as the
// direct form (direct-form re-test, sqrt-sum test, exact integer nint).
#pragma once

#include "tsp2opt_sweep.cuh"

namespace tsp2opt {

constexpr float kXfRel = 3.814697265625e-06f;  // 2^-18
constexpr float kXfNever = -1.0e30f;            // K_r for an impossible row test

template <int R>
struct RowsXF {
    float2 xp[(R + 1) / 2];  // centred x of rows (r, r+1), exact small integers
    float2 yp[(R + 1) / 2];
    float2 qp[(R + 1) / 2];  // fl(x^2 + y^2)
};

template <int R>
struct BoundXF {
    int B;           // accept delta < B (lane-local running bound)
    float a2f;       // column offset a2 = (B - 2) - a1
    float kr[R + 1];  // row constants K_r = S_r (1 + 2^-18) + 2^-18 Q_r + 1  (kXfNever if S_r < 0); kr[R] unused
};

// K_r for bound B from the lane's row edges (shared memory) and row norms.
template <int R>
__device__ __forceinline__ void set_bound_xf(BoundXF<R>& b, const RowsXF<R>& rows, const float* my_rowe, int B)
{
    b.B = B;
    const int c = B - 1;
    const int a1 = (c - 1) >> 1;
    const int a2 = c - 1 - a1;
    b.a2f = (float)a2;
#pragma unroll
    for (int r = 0; r < R; r++) {
        const float t = my_rowe[r] + (float)a1;
        const float q = (r & 1) ? rows.qp[r >> 1].y : rows.qp[r >> 1].x;
        b.kr[r] = t < 0.f ? kXfNever : fmaf(fmaf(t, t, t), 1.f + kXfRel, fmaf(q, kXfRel, 1.f));
    }
    b.kr[R] = kXfNever;
}

// u for one column: two FFMA2 per pair of rows.  m = (-2x'_k, -2x'_k, -2y'_k, -2y'_k).
template <int R>
__device__ __forceinline__ void column_u(float (&u)[R + 1], const RowsXF<R>& rows, float4 m)
{
    const float2 mx = make_float2(m.x, m.y), my = make_float2(m.z, m.w);
#pragma unroll
    for (int q = 0; q < (R + 1) / 2; q++) {
        const float2 v = fma2(rows.xp[q], mx, fma2(rows.yp[q], my, rows.qp[q]));
        u[2 * q] = v.x;
        u[2 * q + 1] = v.y;
    }
}

// min over r < R of u_r - K_r (row test values of this column)
template <int R>
__device__ __forceinline__ float row_min(const float (&u)[R + 1], const BoundXF<R>& b)
{
    float t[R + 1];
#pragma unroll
    for (int q = 0; q < (R + 1) / 2; q++) {
        const float2 v = add2(make_float2(u[2 * q], u[2 * q + 1]), make_float2(-b.kr[2 * q], -b.kr[2 * q + 1]));
        t[2 * q] = v.x;
        t[2 * q + 1] = v.y;
    }
    return tree_min<0, R>(t);
}

// Column data in shared memory (xf layout): m = (-2x', -2x', -2y', -2y') and
// w = (W_k, e_k) with W_k = -Q_k (1 - 2^-18), Q_k = fl(x'^2 + y'^2).
struct TileSmemXF {
    float4* colm;  // [TJ + 2]: columns J0..J1 and one spare
    float2* colw;  // [TJ + 2]
    float* rowe;   // [32 * R * warps]
    __device__ TileSmemXF(void* base, int TJ)
        : colm(reinterpret_cast<float4*>(base)),
          colw(reinterpret_cast<float2*>(colm + TJ + 2)),
          rowe(reinterpret_cast<float*>(colw + TJ + 2))
    {
    }
};

__host__ __device__ inline size_t tile_smem_bytes_xf(int TJ, int TI)
{
    return (size_t)(TJ + 2) * (sizeof(float4) + sizeof(float2)) + (size_t)TI * sizeof(float);
}

// Rare path of the xf walk: re-test this lane's pairs (r, j) with the direct
// form (exact dx, dy; tsp2opt_sweep.cuh), then the sqrt-sum test, then exact.
// Rolled loop over r with the row cities re-read from P (L1) and the row
// edges from shared memory, so the rare path adds no register pressure to the
// fast loop.
template <int R, bool MASK, bool PS>
__device__ __forceinline__ void exact_step_xf(BoundXF<R>& b, const float2* P, int row0, int j, float4 mj, float4 mj1,
                                              float ej, const float* my_rowe, float cxb, float cyb,
                                              unsigned long long& mykey)
{
    const int c = b.B - 1;
    const int a1 = (c - 1) >> 1;
    const float scol = sq_threshold(ej + b.a2f);
    // column cities j, j+1 as biased floats (exact: centred integer + biased centre)
    const float xj = fmaf(-0.5f, mj.x, cxb), yj = fmaf(-0.5f, mj.z, cyb);
    const float xj1 = fmaf(-0.5f, mj1.x, cxb), yj1 = fmaf(-0.5f, mj1.z, cyb);
    const float lim = ej + (float)b.B + 0.5f;
    const int ixj = unbias(xj), iyj = unbias(yj), ixj1 = unbias(xj1), iyj1 = unbias(yj1);
    const int ejn = (int)ej;
    int B = b.B;
    int nexact = 0;
#pragma unroll 1
    for (int r = 0; r < R; r++) {
        if (MASK && row0 + r >= j) break;  // rows ascend: the rest are masked too
        const float2 pr = gld<PS>(P + row0 + r), pr1 = gld<PS>(P + row0 + r + 1);
        const float dx = pr.x - xj, dy = pr.y - yj, dx1 = pr1.x - xj1, dy1 = pr1.y - yj1;  // exact
        const float s1 = fmaf(dx, dx, dy * dy), s2 = fmaf(dx1, dx1, dy1 * dy1);
        const float er = my_rowe[r];
        if (!((s1 <= sq_threshold(er + (float)a1)) || (s2 <= scol))) continue;
        if (!(sqrt_approx(s1) + sqrt_approx(s2) <= er + lim)) continue;
        nexact++;
        const int d = exact_dist_xy(unbias(pr.x), unbias(pr.y), ixj, iyj) +
                      exact_dist_xy(unbias(pr1.x), unbias(pr1.y), ixj1, iyj1) - (int)er - ejn;
        if (d < B) {  // ascending r == ascending cell number
            B = d;
            mykey = pack_key(d, row0 + r, j);
        }
    }
#ifdef TSP2OPT_STATS
    atomicAdd(&g_stats[2], (unsigned long long)nexact);
#endif
    (void)nexact;
    b.B = B;
}

template <int R, bool MASK, bool PS>
__device__ __forceinline__ void walk_xf(const RowsXF<R>& rows, BoundXF<R>& b, int row0, int jstart, int J0, int J1,
                                        const TileSmemXF& sm, const float* my_rowe, float qmarg, float cxb, float cyb,
                                        const float2* P, unsigned long long& mykey)
{
    float ua[R + 1], ub[R + 1];
    const unsigned am = smem_addr(sm.colm) - 16u * (unsigned)J0;  // &colm[j] = am + 16 j
    const unsigned aw = smem_addr(sm.colw) - 8u * (unsigned)J0;   // &colw[j] = aw + 8 j
    float4 mj = lds4(am + 16u * jstart);
    float2 wj = lds2(aw + 8u * jstart);
    column_u<R>(ua, rows, mj);
    float mtj = row_min<R>(ua, b);  // row-test value of column j
    auto step = [&](const float (&cur)[R + 1], float (&nxt)[R + 1], int j) {
        const float4 mj1 = lds4(am + 16u * (j + 1));
        const float2 wj1 = lds2(aw + 8u * (j + 1));
        column_u<R>(nxt, rows, mj1);
        const float ej = wj.y;
        const float T = sq_threshold(ej + b.a2f) * (1.f + kXfRel) + (wj1.x + qmarg);
        bool any;
        float mtn;
        if (!MASK) {
            const float mu = tree_min<1, R + 1>(nxt);
            mtn = row_min<R>(nxt, b);
            any = (mu <= T) || (mtj <= wj.x);
        } else {
            any = false;
#pragma unroll
            for (int r = 0; r < R; r++)
                any |= ((cur[r] - b.kr[r] <= wj.x) || (nxt[r + 1] <= T)) && (row0 + r < j);
            mtn = 0.f;
        }
#ifdef TSP2OPT_STATS
        if ((threadIdx.x & 31) == 0) atomicAdd(&g_stats[0], 1ULL);
#endif
        if (__builtin_expect(__any_sync(0xffffffffu, any), 0)) {
#ifdef TSP2OPT_STATS
            if ((threadIdx.x & 31) == 0) atomicAdd(&g_stats[1], 1ULL);
#endif
            const int B0 = b.B;
            if (any) exact_step_xf<R, MASK, PS>(b, P, row0, j, mj, mj1, ej, my_rowe, cxb, cyb, mykey);
            const int wb = __reduce_min_sync(0xffffffffu, b.B);
            const int nb = min(b.B, wb + 1);
            if (nb < B0) {
                set_bound_xf<R>(b, rows, my_rowe, nb);
                if (!MASK) mtn = row_min<R>(nxt, b);
            }
        }
        mtj = mtn;
        mj = mj1;
        wj = wj1;
    };
    int j = jstart;
    for (; j + 1 < J1; j += 2) {
        step(ua, ub, j);
        step(ub, ua, j + 1);
    }
    if (j < J1) step(ua, ub, j);
}

// Unmasked walk, software-pipelined: the u values of column j+2 (two FFMA2 per
// row pair, then their two minima) are computed in the same basic block as the
// tests of step j, before step j's warp-uniform branch, so the FMA chains of
// the next column overlap the min trees and the vote of the current one.  Only
// scalars cross iterations: mt (row-test minimum of a column), mu (column-test
// minimum of the next column) and (W, e) of the column.  The shared chunk
// holds one spare column past J1 so the last prefetch needs no guard.
template <int R, bool PS>
__device__ __forceinline__ void walk_xf_pipelined(const RowsXF<R>& rows, BoundXF<R>& b, int row0, int jstart,
                                                  int J0, int J1, const TileSmemXF& sm, const float* my_rowe,
                                                  float qmarg, float cxb, float cyb, const float2* P,
                                                  unsigned long long& mykey)
{
    const unsigned am = smem_addr(sm.colm) - 16u * (unsigned)J0;  // &colm[j] = am + 16 j
    const unsigned aw = smem_addr(sm.colw) - 8u * (unsigned)J0;   // &colw[j] = aw + 8 j
    float u[R + 1];
    column_u<R>(u, rows, lds4(am + 16u * jstart));
    float mt0 = row_min<R>(u, b);                 // row test, column j
    column_u<R>(u, rows, lds4(am + 16u * (jstart + 1)));
    float mu0 = tree_min<1, R + 1>(u);            // column test of step j (column j+1)
    float mt1 = row_min<R>(u, b);                 // row test, column j+1
    float2 w0 = lds2(aw + 8u * jstart), w1 = lds2(aw + 8u * (jstart + 1));
#pragma unroll 2
    for (int j = jstart; j < J1; j++) {
        // next column's work first (independent of this step's branch)
        const float2 w2 = lds2(aw + 8u * (j + 2));
        column_u<R>(u, rows, lds4(am + 16u * (j + 2)));
        const float mu1 = tree_min<1, R + 1>(u);
        const float mt2 = row_min<R>(u, b);
        // this step's tests
        const float T = sq_threshold(w0.y + b.a2f) * (1.f + kXfRel) + (w1.x + qmarg);
        const bool any = (mu0 <= T) || (mt0 <= w0.x);
#ifdef TSP2OPT_STATS
        if ((threadIdx.x & 31) == 0) atomicAdd(&g_stats[0], 1ULL);
#endif
        if (__builtin_expect(__any_sync(0xffffffffu, any), 0)) {
#ifdef TSP2OPT_STATS
            if ((threadIdx.x & 31) == 0) atomicAdd(&g_stats[1], 1ULL);
#endif
            const int B0 = b.B;
            if (any)
                exact_step_xf<R, false, PS>(b, P, row0, j, lds4(am + 16u * j), lds4(am + 16u * (j + 1)), w0.y,
                                            my_rowe, cxb, cyb, mykey);
            const int wb = __reduce_min_sync(0xffffffffu, b.B);
            const int nb = min(b.B, wb + 1);
            if (nb < B0) set_bound_xf<R>(b, rows, my_rowe, nb);  // mt1/mt2 stay looser: still sound
        }
        mt0 = mt1;
        mt1 = mt2;
        mu0 = mu1;
        w0 = w1;
        w1 = w2;
    }
}

template <int R, bool PS>
__device__ __forceinline__ void sweep_tile_xf(const float2* P, const int* E, int n, int2 tile, int TJ, Slot* slot,
                                              const TileSmemXF& sm)
{
    const int I0 = tile.x, J0 = tile.y;
    const int J1 = min(J0 + TJ, n);
    const int ncol = J1 - J0;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int wrow0 = I0 + warp * 32 * R;
    const int row0 = wrow0 + lane * R;
    const int jstart = max(J0, wrow0 + 1);
    const bool active = jstart < J1;
    float* my_rowe = sm.rowe + threadIdx.x * R;
    const float2 ctr = gld<PS>(P + I0);  // tile centre (biased floats of city I0)

    RowsXF<R> rows;
    int erow[R];
    float qmax = 0.f;
    if (active) {
#pragma unroll
        for (int q = 0; q < (R + 1) / 2; q++) {
            const float2 p0 = gld<PS>(P + row0 + 2 * q), p1 = gld<PS>(P + row0 + 2 * q + 1);
            rows.xp[q] = make_float2(p0.x - ctr.x, p1.x - ctr.x);  // exact
            rows.yp[q] = make_float2(p0.y - ctr.y, p1.y - ctr.y);
        }
#pragma unroll
        for (int r = 0; r < R; r++) erow[r] = gld<PS>(E + row0 + r);
#pragma unroll
        for (int q = 0; q < (R + 1) / 2; q++) {
            rows.qp[q] = fma2(rows.xp[q], rows.xp[q], mul2(rows.yp[q], rows.yp[q]));
            qmax = fmaxf(qmax, fmaxf(rows.qp[q].x, rows.qp[q].y));
        }
    }
    for (int c = threadIdx.x; c <= ncol + 1; c += blockDim.x) {  // + 1 spare column (pipelined prefetch)
        const float2 p = gld<PS>(P + J0 + c);
        const int e = gld<PS>(E + J0 + c);
        const float x = p.x - ctr.x, y = p.y - ctr.y;
        const float q = fmaf(x, x, y * y);
        sm.colm[c] = make_float4(-2.f * x, -2.f * x, -2.f * y, -2.f * y);
        sm.colw[c] = make_float2(-q * (1.f - kXfRel), (float)e);
    }
    const int dg = key_delta(*(volatile unsigned long long*)&slot->key);
    if (active) {
#pragma unroll
        for (int r = 0; r < R; r++) my_rowe[r] = (float)erow[r];
    }
    __syncthreads();
    if (!active) return;

    unsigned long long mykey = kKeyNone;
    BoundXF<R> b;
    set_bound_xf<R>(b, rows, my_rowe, dg == 0 ? 0 : dg + 1);
    const float qmarg = fmaf(qmax, kXfRel, 1.f);  // row-side margin of the column test
    const bool masked = (wrow0 + 32 * R - 1) >= jstart;
    if (masked) walk_xf<R, true, PS>(rows, b, row0, jstart, J0, J1, sm, my_rowe, qmarg, ctr.x, ctr.y, P, mykey);
    else walk_xf_pipelined<R, PS>(rows, b, row0, jstart, J0, J1, sm, my_rowe, qmarg, ctr.x, ctr.y, P, mykey);

#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const unsigned long long other = __shfl_xor_sync(0xffffffffu, mykey, o);
        mykey = other < mykey ? other : mykey;
    }
    if (lane == 0 && mykey < *(volatile unsigned long long*)&slot->key) atomicMin(&slot->key, mykey);
}

}  // namespace tsp2opt
