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

namespace tsp2opt {

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
}

__global__ void reset_key_kernel(Slot* slot) { slot->key = seed_key(); }

// ===========================================================================
// a4 + a5: the sweep.  One CTA = one tile = rows [I0, I0 + 32*R*NW) x columns
// [J0, J0 + TJ).  Each lane owns R consecutive rows (R+1 cities in registers),
// the warp walks the tile's columns; column city j is a shared-memory broadcast.
// Per column step the lane computes the R+1 squared distances of its rows to
// column j+1 (diagonal reuse: s(i+1, j+1) of pair (i, j) is s(i', j') of pair
// (i', j') = (i+1, j+1)), and tests every pair (i, j) with the exact
// necessary condition of DESIGN.md §5.2:
//     delta(i,j) <= B - 1   ==>   D(i,j) <= e_i + a1   or   D(i+1,j+1) <= e_j + a2
// (a1 + a2 = B - 2), evaluated on squared distances (no sqrt).  Pairs that pass
// are evaluated exactly (integer nint, same as the oracle) and accepted iff
// delta < B; B is the lane's running bound, started from the global best.
// Pairs are visited in increasing Fig. 3 cell order per lane, so a strict '<'
// keeps the lowest cell among equal deltas (reading R5).
// ===========================================================================
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
    int B;      // accept delta < B (lane-local running bound)
    float a2f;  // column offset a2 = (B - 2) - a1
    float srow[R];  // row thresholds: D(i_r, j) <= e_{i_r} + a1  <=>  s <= srow[r]
};

// Thresholds of the exact necessary condition for bound B:
// delta <= B - 1 = c  ==>  D(i,j) <= e_i + a1  or  D(i+1,j+1) <= e_j + a2,
// a1 = floor((c - 1) / 2), a2 = c - 1 - a1.  Row edges are re-read from E
// (L1-resident; this runs once per tile and when B drops).
template <int R>
__device__ __forceinline__ void set_bound(Bound<R>& b, const int* __restrict__ E, int row0, int B)
{
    b.B = B;
    const int c = B - 1;
    const int a1 = (c - 1) >> 1;
    const int a2 = c - 1 - a1;
    b.a2f = (float)a2;
#pragma unroll
    for (int r = 0; r < R; r++) b.srow[r] = sq_threshold((float)(E[row0 + r] + a1));
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
            const bool t = cur[r] <= b.srow[r];
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
// only lanes with a candidate run it).  Integer nint distances, identical
// arithmetic to the oracle; accept delta < B in increasing cell order.
template <int R, bool MASK>
__device__ __forceinline__ void exact_step(Bound<R>& b, const float (&cur)[R + 1], const float (&nxt)[R + 1],
                                           float scol, int row0, int j, float4 c0, float4 c1, float ej,
                                           const float2* __restrict__ P, const int* __restrict__ E,
                                           unsigned long long& mykey)
{
    unsigned mask = 0;
#pragma unroll
    for (int r = 0; r < R; r++) {
        bool cand = (cur[r] <= b.srow[r]) || (nxt[r + 1] <= scol);
        if (MASK) cand = cand && (row0 + r < j);
        mask |= (cand ? 1u : 0u) << r;
    }
    const int xj = unbias(-c0.x), yj = unbias(-c0.z);
    const int xj1 = unbias(-c1.x), yj1 = unbias(-c1.z);
    const int ejn = (int)ej;
    int B = b.B;
    while (mask) {  // ascending r == ascending cell number
        const int r = __ffs(mask) - 1;
        mask &= mask - 1;
        const float2 pi = P[row0 + r], pi1 = P[row0 + r + 1];
        const int d = exact_dist_xy(unbias(pi.x), unbias(pi.y), xj, yj) +
                      exact_dist_xy(unbias(pi1.x), unbias(pi1.y), xj1, yj1) - E[row0 + r] - ejn;
        if (d < B) {
            B = d;
            mykey = pack_key(d, row0 + r, j);
        }
    }
    b.B = B;
}

template <int R, bool MASK>
__device__ __forceinline__ void column_step(const Rows<R>& rows, Bound<R>& b, const float (&cur)[R + 1],
                                            float (&nxt)[R + 1], int row0, int j, int J0,
                                            const float4* __restrict__ colxy, const float* __restrict__ cole,
                                            const float2* __restrict__ P, const int* __restrict__ E,
                                            unsigned long long& mykey)
{
    const float4 c1 = colxy[j + 1 - J0];
    column_sq<R>(nxt, rows, c1);
    const float ej = cole[j - J0];
    const float scol = sq_threshold(ej + b.a2f);
    const bool any = step_any<R, MASK>(b, cur, nxt, scol, row0, j);
    if (__builtin_expect(__any_sync(0xffffffffu, any), 0)) {
        const int B0 = b.B;
        if (any) exact_step<R, MASK>(b, cur, nxt, scol, row0, j, colxy[j - J0], c1, ej, P, E, mykey);
        // share the warp's best: a lane may accept delta <= (best of another lane)
        const int wb = __reduce_min_sync(0xffffffffu, b.B);
        const int nb = min(b.B, wb + 1);
        if (nb < B0) set_bound<R>(b, E, row0, nb);
    }
}

template <int R, bool MASK>
__device__ __forceinline__ void walk(const Rows<R>& rows, Bound<R>& b, int row0, int jstart, int J0, int J1,
                                     const float4* __restrict__ colxy, const float* __restrict__ cole,
                                     const float2* __restrict__ P, const int* __restrict__ E,
                                     unsigned long long& mykey)
{
    float sa[R + 1], sb[R + 1];
    column_sq<R>(sa, rows, colxy[jstart - J0]);
    int j = jstart;
    for (; j + 1 < J1; j += 2) {
        column_step<R, MASK>(rows, b, sa, sb, row0, j, J0, colxy, cole, P, E, mykey);
        column_step<R, MASK>(rows, b, sb, sa, row0, j + 1, J0, colxy, cole, P, E, mykey);
    }
    if (j < J1) column_step<R, MASK>(rows, b, sa, sb, row0, j, J0, colxy, cole, P, E, mykey);
}

template <int R>
__global__ void __launch_bounds__(128) sweep_kernel(const float2* __restrict__ P, const int* __restrict__ E, int n,
                                                     const int2* __restrict__ tiles, int TJ, Slot* __restrict__ slot,
                                                     int respect_done)
{
    extern __shared__ float4 smem[];
    float4* colxy = smem;                                    // [TJ + 1]: (-x, -x, -y, -y) of columns J0..J1
    float* cole = reinterpret_cast<float*>(smem + TJ + 1);  // [TJ + 1]: e_j as float

    if (respect_done && *(volatile int*)&slot->done) return;  // converged: iteration is a no-op
    const int2 tile = tiles[blockIdx.x];
    const int I0 = tile.x, J0 = tile.y;
    const int J1 = min(J0 + TJ, n);  // columns j in [J0, J1), j <= n-1
    const int ncol = J1 - J0;
    for (int c = threadIdx.x; c <= ncol; c += blockDim.x) {  // J1 <= n: P[n] = P[0] closes the tour
        const float2 p = P[J0 + c];
        colxy[c] = make_float4(-p.x, -p.x, -p.y, -p.y);
        cole[c] = (float)E[J0 + c];
    }
    __syncthreads();

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int wrow0 = I0 + warp * 32 * R;
    const int row0 = wrow0 + lane * R;
    const int jstart = max(J0, wrow0 + 1);  // no pair of this warp has j <= wrow0
    if (jstart >= J1) return;                // warp-uniform: nothing to do
    unsigned long long mykey = kKeyNone;
    Rows<R> rows;
#pragma unroll
    for (int q = 0; q < (R + 1) / 2; q++) {
        const float2 p0 = P[row0 + 2 * q], p1 = P[row0 + 2 * q + 1];
        rows.xp[q] = make_float2(p0.x, p1.x);
        rows.yp[q] = make_float2(p0.y, p1.y);
    }
    // Start from the best key any CTA of this sweep has published so far.  The
    // slot key is the seed (0, cell 0) or a real pair of this sweep, so a pair of
    // ours can only win with delta < 0 (key delta 0) or delta <= key delta.
    const unsigned long long g = *(volatile unsigned long long*)&slot->key;
    const int dg = key_delta(g);
    Bound<R> b;
    set_bound<R>(b, E, row0, dg == 0 ? 0 : dg + 1);
    const bool masked = (wrow0 + 32 * R - 1) >= jstart;  // warp-uniform: some row >= some j
    if (masked) walk<R, true>(rows, b, row0, jstart, J0, J1, colxy, cole, P, E, mykey);
    else walk<R, false>(rows, b, row0, jstart, J0, J1, colxy, cole, P, E, mykey);

    // a5: warp min, one atomicMin per warp (L16 Fig. 4 "Get best local pair ...
    // Get best global pair"); min is order-independent -> deterministic result.
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const unsigned long long other = __shfl_xor_sync(0xffffffffu, mykey, o);
        mykey = other < mykey ? other : mykey;
    }
    if (lane == 0 && mykey < *(volatile unsigned long long*)&slot->key) atomicMin(&slot->key, mykey);
}

// ===========================================================================
// a7 + a8: apply the best move of slot_in (or an explicit (i, j)) and write
// the next iteration's state into slot_out.  Reverses P and tour on [i+1, j]
// and e on [i+1, j-1]; the two new edges are exact distances of the
// pre-reversal cities (thread 0 reads them before doing its own swap; no other
// thread touches P[i], P[i+1], P[j], P[j+1], e[i], e[j]).
// ===========================================================================
__global__ void __launch_bounds__(256) apply_kernel(float2* __restrict__ P, int* __restrict__ E, int* __restrict__ tour,
                                                    const Slot* __restrict__ in, Slot* __restrict__ out,
                                                    long long max_moves, int explicit_move, int ei, int ej)
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
    const int gtid = blockIdx.x * blockDim.x + threadIdx.x;
    const int stride = gridDim.x * blockDim.x;
    if (gtid == 0) {
        Slot o;
        o.key = seed_key();
        o.last_key = explicit_move ? in->last_key : key;
        o.moves = moves;
        o.length = in->length;
        o.done = done;
        if (!explicit_move && !done) {
            if (key_delta(key) >= 0) o.done = 1;        // local minimum (reading R7)
            else if (moves >= max_moves) o.done = 2;    // capped with an improving move left (R8)
        }
        if (apply) {
            const float2 pi = P[i], pj = P[j], pi1 = P[i + 1], pj1 = P[j + 1];
            const int ni = exact_dist_biased(pi, pj), nj = exact_dist_biased(pi1, pj1);
            o.length += (long long)ni + nj - E[i] - E[j];
            o.moves = moves + 1;
            E[i] = ni;
            E[j] = nj;
        }
        *out = o;
    }
    if (!apply) return;
    const int half = (j - i) >> 1;  // swap P/tour positions i+1+t <-> j-t
    for (int t = gtid; t < half; t += stride) {
        const int a = i + 1 + t, c = j - t;
        const float2 pa = P[a], pc = P[c];
        P[a] = pc;
        P[c] = pa;
        const int ta = tour[a], tc = tour[c];
        tour[a] = tc;
        tour[c] = ta;
    }
    const int ehalf = (j - i - 1) >> 1;  // swap e positions i+1+t <-> j-1-t
    for (int t = gtid; t < ehalf; t += stride) {
        const int a = i + 1 + t, c = j - 1 - t;
        const int ea = E[a], ec = E[c];
        E[a] = ec;
        E[c] = ea;
    }
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
        if (!(s.x <= S) || !(s.y <= S)) {
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
long long launch_count() { return g_launches.load(); }

cudaError_t launch_load_tour(const int* coords, const int* tour_src, int* tour_dst, float2* P, int* E, int n,
                             Slot* slot, unsigned* stamp, unsigned epoch, cudaStream_t st)
{
    init_slot_kernel<<<1, 1, 0, st>>>(slot, 1);
    load_tour_kernel<<<(n + 255) / 256, 256, 0, st>>>(coords, tour_src, tour_dst, P, E, n, slot, stamp, epoch);
    g_launches += 2;
    return cudaGetLastError();
}

cudaError_t launch_reset_key(Slot* slot, cudaStream_t st)
{
    reset_key_kernel<<<1, 1, 0, st>>>(slot);
    g_launches += 1;
    return cudaGetLastError();
}

size_t sweep_smem_bytes(int TJ) { return (size_t)(TJ + 1) * sizeof(float4) + (size_t)(TJ + 1) * sizeof(float); }

cudaError_t sweep_prepare()
{
    return cudaFuncSetAttribute(sweep_kernel<kRows>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)sweep_smem_bytes(kMaxTJ));
}

cudaError_t launch_sweep(const Geometry& g, const float2* P, const int* E, int n, const int2* tiles, int ntiles,
                         Slot* slot, int respect_done, cudaStream_t st)
{
    if (ntiles <= 0) return cudaSuccess;
    sweep_kernel<kRows><<<ntiles, 32 * g.warps, sweep_smem_bytes(g.tj), st>>>(P, E, n, tiles, g.tj, slot,
                                                                               respect_done);
    g_launches += 1;
    return cudaGetLastError();
}

cudaError_t launch_apply(float2* P, int* E, int* tour, int n, const Slot* in, Slot* out, long long max_moves,
                         int explicit_move, int ei, int ej, cudaStream_t st)
{
    int blocks = (n / 2 + 255) / 256;
    if (blocks < 1) blocks = 1;
    if (blocks > 4 * 148) blocks = 4 * 148;
    apply_kernel<<<blocks, 256, 0, st>>>(P, E, tour, in, out, max_moves, explicit_move, ei, ej);
    g_launches += 1;
    return cudaGetLastError();
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
