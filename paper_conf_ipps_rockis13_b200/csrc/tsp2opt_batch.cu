// tsp2opt_batch.cu -- many independent small instances, one CTA each
// ("Batched small-instance sweeps ... one CTA each";
// the paper's small-n weakness, L18 §V "the GPU ILS version does not give any
// substantial speedup ... in case of small problems (smaller than 200)").
//
// Each CTA runs the whole best-improvement local search of its instance in
// shared memory: route-ordered coordinates, tour and edges never leave the SM.
// A sweep walks the C(n,2) pairs diagonal by diagonal (g = j - i): warps take
// diagonals longest-first in a snake order and cover each in
// 31-pair windows: lane l computes the float distance D(i0+l, i0+l+g) and
// takes D(i0+l+1, i0+l+1+g) from lane l+1 by shuffle (conflict-free shared
// loads, one MUFU.SQRT per pair).  Only pairs whose float delta lies within
// the DESIGN.md §5.8 error bound of the best delta found so far in this sweep
// (shared by the block) get exact EUC_2D distances and a packed (delta, j, i)
// key; a block-wide min picks the move (lowest delta, then lowest Fig. 3 cell
// -- reading R5) and the block reverses positions i+1..j in place.  Two
// __syncthreads per move.  Same results as tsp2opt_local_search / the oracle,
// instance by instance.
#include <cstdlib>

#include "tsp2opt_device.cuh"
#include "tsp2opt_internal.h"

namespace tsp2opt {

constexpr int kBatchMaxThreads = 256;
constexpr int kBatchPackedMaxN = 256;  // measured: packed wins at n = 100, ties at 200, loses at 1002

// Exact-test margin of the float filter: with a relative
// MUFU.SQRT error <= 2^-21 (tsp2opt_selftest_sqrt) and s_f within 2^-23 of s,
// |r - sqrt(s)| <= 0.025 for every reachable s, so nint(sqrt(s)) >= r - 0.525
// per distance, and the float delta (three roundings <= 0.008 each) exceeds the
// exact one by at most 1.074.  delta <= B therefore implies df <= B + 1.25.
constexpr float kBatchSlack = 1.25f;
constexpr long long kNoMoveCap = 0x7FFFFFFFFFFFFFFFLL;

// Shared state of one CTA's local search.
struct BlockLs {
    unsigned long long red[2][kBatchMaxThreads / 32];
    long long len;  // current tour length
    int bad;
    int best[2];    // per-sweep shared bound (ping-pong)
};

// Best-improvement local search of the CTA's instance, in shared memory:
// P[n+1] / E[n+1] / tour[n] hold a loaded tour and ls.len its length.  Runs
// to the local minimum or max_iters moves; returns the moves applied.  All
// threads of the CTA call it; it ends with a __syncthreads.
template <bool PACKED>
__device__ __forceinline__ long long block_local_search(float2* P, float* E, int* tour, int n, long long max_iters, BlockLs& ls)
{
    const int T = blockDim.x, nw = T >> 5, lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    // packed layout: this warp's windows and its lane's first entry
    int pk0 = 0, pk1 = 0, pi0 = 0, plim0 = 0;
    if (PACKED) {
        const int Mx = n * (n - 1) / 2 + (n - 1);  // pairs + one sentinel entry per diagonal
        const int nwin = (Mx + 30) / 31, wper = (nwin + nw - 1) / nw;
        pk0 = min(nwin, wper * w);
        pk1 = min(nwin, pk0 + wper);
        int q = 31 * pk0 + lane;
        plim0 = n - 1;
        while (q > plim0 && plim0 > 0) {
            q -= plim0 + 1;
            plim0--;
        }
        pi0 = q;
    }
    if (threadIdx.x == 0) ls.best[0] = ls.best[1] = 0;
    __syncthreads();

    long long moves = 0;
    for (int par = 0;; par ^= 1) {
        unsigned long long key = seed_key();
        float Bl = lane == 31 ? -1e30f : kBatchSlack;  // lane 31 only feeds its distance to lane 30
        if (PACKED) {
            // one stream of distance entries, diagonal after diagonal (diagonal
            // g = n - lim holds entries i = 0 .. lim), cut into 31-pair windows;
            // warp w owns windows [k0, k1).  A lane wraps to the next diagonal
            // in place; past the last diagonal it idles on entry (0, n).
            int i = pi0, lim = plim0;
            int since = 0;
#pragma unroll 1
            for (int k = pk0; k < pk1; k++) {
                const int g = n - lim;
                const int ic = min(i, lim);
                const float2 pa = P[ic], pc = P[ic + g];
                const float dx = pa.x - pc.x, dy = pa.y - pc.y;
                const float rr = sqrt_approx(fmaf(dx, dx, dy * dy));
                const float rn = __shfl_down_sync(0xffffffffu, rr, 1);
                const float df = ((rr + rn) - E[ic]) - E[ic + g];
                const bool cand = i < lim && df <= Bl;
                if (__ballot_sync(0xffffffffu, cand)) {  // rare: exact delta and key
                    if (cand) {
                        const int d = exact_dist_biased(pa, pc) + exact_dist_biased(P[i + 1], P[i + 1 + g]) -
                                      (int)E[i] - (int)E[i + g];
                        const unsigned long long kk = pack_key(d, i, i + g);
                        key = kk < key ? kk : key;
                    }
                    since = 8;
                }
                if (++since >= 8) {  // share the best delta with the block (see below)
                    since = 0;
                    const int Bw = __reduce_min_sync(0xffffffffu, key_delta(key));
                    const int Bs = *(volatile int*)&ls.best[par];
                    if (Bw < Bs && lane == 0) atomicMin(&ls.best[par], Bw);
                    if (lane != 31) Bl = (float)min(Bw, Bs) + kBatchSlack;
                }
                i += 31;
                while (i > lim && lim > 0) {
                    i -= lim + 1;
                    lim--;
                }
            }
        } else {
            // diagonals dealt to warps in a snake order (round r: w, or nw-1-w when r
            // is odd) so the longest-first lengths balance without a shared counter
            for (int r = 0;; r++) {
                const int g = 1 + r * nw + ((r & 1) ? nw - 1 - w : w);
                if (g >= n) break;
                const int lim = n - g;  // pairs i = 0 .. lim-1, distance entries i = 0 .. lim
                const float2* Pg = P + g;
                const float* Eg = E + g;
                bool hit = false;
    #pragma unroll 1
                for (int i = lane; i - lane < lim; i += 31) {
                    const int ic = min(i, lim);
                    const float2 pa = P[ic], pc = Pg[ic];
                    const float dx = pa.x - pc.x, dy = pa.y - pc.y;
                    const float r = sqrt_approx(fmaf(dx, dx, dy * dy));
                    const float rn = __shfl_down_sync(0xffffffffu, r, 1);
                    const float df = ((r + rn) - E[ic]) - Eg[ic];
                    const bool cand = i < lim && df <= Bl;
                    if (__ballot_sync(0xffffffffu, cand)) {  // rare: exact delta and key
                        if (cand) {
                            const int d = exact_dist_biased(pa, pc) + exact_dist_biased(P[i + 1], Pg[i + 1]) -
                                          (int)E[i] - (int)Eg[i];
                            const unsigned long long kk = pack_key(d, i, i + g);
                            key = kk < key ? kk : key;
                        }
                        const int Bw = __reduce_min_sync(0xffffffffu, key_delta(key));
                        if (lane != 31) Bl = (float)Bw + kBatchSlack;
                        hit = true;
                    }
                }
                // share the warp's best delta with the block (any attained delta
                // bounds the sweep's min): publish after a hit, poll every 4th diagonal
                if (hit || (r & 3) == 3) {
                    const int Bw = __reduce_min_sync(0xffffffffu, key_delta(key));
                    const int Bs = *(volatile int*)&ls.best[par];
                    if (Bw < Bs && lane == 0) atomicMin(&ls.best[par], Bw);
                    if (lane != 31) Bl = (float)min(Bw, Bs) + kBatchSlack;
                }
            }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            const unsigned long long v = __shfl_xor_sync(0xffffffffu, key, o);
            key = v < key ? v : key;
        }
        if (lane == 0) ls.red[par][w] = key;
        __syncthreads();  // all scans done: P/E may now change; ls.red[par] complete
        unsigned long long best = ls.red[par][0];
        for (int t = 1; t < nw; t++) best = ls.red[par][t] < best ? ls.red[par][t] : best;
        if (threadIdx.x == 0) ls.best[par ^ 1] = 0;  // the next sweep's bound (read after the closing barrier)
        if (key_delta(best) >= 0 || moves >= max_iters) break;
        // reverse positions i+1..j of P and tour, edges on [i+1, j-1]; thread 0
        // owns the swap of (i+1, j), so it reads the old endpoints before writing
        const int bi = key_i(best), bj = key_j(best);
        if (threadIdx.x == 0) {
            const float2 pi = P[bi], pj = P[bj], pi1 = P[bi + 1], pj1 = P[bj + 1];
            E[bi] = (float)exact_dist_biased(pi, pj);
            E[bj] = (float)exact_dist_biased(pi1, pj1);
            ls.len += key_delta(best);
        }
        for (int t = threadIdx.x; t < (bj - bi) / 2; t += T) {
            const int a = bi + 1 + t, c = bj - t;
            const float2 pa = P[a];
            P[a] = P[c];
            P[c] = pa;
            const int ta = tour[a];
            tour[a] = tour[c];
            tour[c] = ta;
        }
        for (int t = threadIdx.x; t < (bj - bi - 1) / 2; t += T) {
            const int a = bi + 1 + t, c = bj - 1 - t;
            const float ea = E[a];
            E[a] = E[c];
            E[c] = ea;
        }
        moves++;
        __syncthreads();
    }
    return moves;
}

// Load instance b (coordinates -> biased P, validated tour) into shared
// memory and compute its edges and length.  Returns false (and reports
// lengths[b] = iters[b] = -1) if the tour is not a permutation or a
// coordinate is out of range.
__device__ __forceinline__ bool block_load(const int* xy, const int* gt, int n, float2* P, float* E, int* tour, BlockLs& ls)
{
    const int T = blockDim.x;
    int* stamp = reinterpret_cast<int*>(E);
    for (int k = threadIdx.x; k <= n; k += T) stamp[k] = 0;
    if (threadIdx.x == 0) {
        ls.bad = 0;
        ls.len = 0;
        ls.best[0] = ls.best[1] = 0;
    }
    __syncthreads();
    for (int k = threadIdx.x; k < n; k += T) {
        const int c = gt[k];
        if (c < 0 || c >= n || atomicAdd(&stamp[c], 1) != 0) {
            ls.bad = 1;
            continue;
        }
        const int x = xy[2 * c], y = xy[2 * c + 1];
        if ((unsigned)x >= (1u << 15) || (unsigned)y >= (1u << 15)) ls.bad = 1;
        tour[k] = c;
        P[k] = make_float2(bias_coord(x), bias_coord(y));
    }
    __syncthreads();
    if (ls.bad) return false;  // uniform
    if (threadIdx.x == 0) P[n] = P[0];
    __syncthreads();
    long long part = 0;
    for (int k = threadIdx.x; k <= n; k += T) {
        const int e = k < n ? exact_dist_biased(P[k], P[k + 1]) : 0;
        E[k] = (float)e;
        part += e;
    }
    atomicAdd((unsigned long long*)&ls.len, (unsigned long long)part);
    __syncthreads();
    return true;
}

template <bool PACKED>
__global__ void __launch_bounds__(kBatchMaxThreads) batch_ls_kernel(const int* __restrict__ coords,
                                                                    int* __restrict__ tours, int n,
                                                                    long long max_iters,
                                                                    long long* __restrict__ lengths,
                                                                    long long* __restrict__ iters)
{
    extern __shared__ float2 bsm[];
    float2* P = bsm;                                  // [n + 1] route-ordered, biased; P[n] = P[0]
    float* E = reinterpret_cast<float*>(P + n + 1);  // [n + 1] e_k = d(k, k+1) (exact integers); E[n] pad
    int* tour = reinterpret_cast<int*>(E + n + 1);    // [n]
    __shared__ BlockLs ls;
    const int b = blockIdx.x;
    int* gt = tours + (long long)n * b;
    if (!block_load(coords + 2LL * n * b, gt, n, P, E, tour, ls)) {
        if (threadIdx.x == 0) lengths[b] = iters[b] = -1;
        return;
    }
    const long long moves = block_local_search<PACKED>(P, E, tour, n, max_iters, ls);
    for (int k = threadIdx.x; k < n; k += blockDim.x) gt[k] = tour[k];
    if (threadIdx.x == 0) {
        lengths[b] = ls.len;
        iters[b] = moves;
    }
}

// Batched Iterated Local Search (L10 Algorithm 1; SURVEY §8(f) NEXT-2
// "batched multi-replica runs for n < 200"): one CTA per replica runs the
// whole of Algorithm 1 in shared memory -- s* = LS(s0); `iterations` times
// {s' = double_bridge(s*, cuts(seeds[b], t)); s*' = LS(s'); s* = s*' iff
// strictly shorter} (readings R14-R16, the same cuts as tsp2opt_ils).
// history (or NULL): int64[batch * (iterations + 1)], the best length after
// each step.  The replica's coordinates are kept in shared memory by city id
// for the re-gather after each perturbation.
template <bool PACKED>
__global__ void __launch_bounds__(kBatchMaxThreads) batch_ils_kernel(const int* __restrict__ coords,
                                                                     int* __restrict__ tours, int n,
                                                                     long long iterations,
                                                                     const unsigned long long* __restrict__ seeds,
                                                                     long long* __restrict__ lengths,
                                                                     long long* __restrict__ history)
{
    extern __shared__ float2 bsm[];
    float2* P = bsm;                                  // [n + 1]
    float* E = reinterpret_cast<float*>(P + n + 1);  // [n + 1]
    int* tour = reinterpret_cast<int*>(E + n + 1);    // [n] current tour
    int* best = tour + n;                             // [n] s*
    float2* C = reinterpret_cast<float2*>((reinterpret_cast<uintptr_t>(best + n) + 7) & ~uintptr_t(7));  // [n] by city id
    __shared__ BlockLs ls;
    __shared__ long long s_best_len;
    const int b = blockIdx.x, T = blockDim.x;
    const int* xy = coords + 2LL * n * b;
    int* gt = tours + (long long)n * b;
    long long* hist = history ? history + (iterations + 1) * b : nullptr;
    if (!block_load(xy, gt, n, P, E, tour, ls)) {
        if (threadIdx.x == 0) lengths[b] = -1;
        return;
    }
    for (int c = threadIdx.x; c < n; c += T) C[c] = make_float2(bias_coord(xy[2 * c]), bias_coord(xy[2 * c + 1]));
    block_local_search<PACKED>(P, E, tour, n, kNoMoveCap, ls);
    for (int k = threadIdx.x; k < n; k += T) best[k] = tour[k];
    if (threadIdx.x == 0) {
        s_best_len = ls.len;
        if (hist) hist[0] = ls.len;
    }
    __syncthreads();
    const unsigned long long seed = seeds[b];
    for (long long t = 0; t < iterations; t++) {
        if (n >= 8) {
            long long a, bb, c;
            ils_cuts(n, seed, t, &a, &bb, &c);
            // s' = A C B D of s* = A B C D, gathered with its coordinates and edges
            for (int k = threadIdx.x; k < n; k += T) {
                int src;
                if (k < a || k >= c) src = k;
                else if (k < a + (c - bb)) src = (int)(bb + (k - a));
                else src = (int)(a + (k - a - (c - bb)));
                const int city = best[src];
                tour[k] = city;
                P[k] = C[city];
            }
            if (threadIdx.x == 0) ls.len = 0;
            __syncthreads();
            if (threadIdx.x == 0) P[n] = P[0];
            __syncthreads();
            long long part = 0;
            for (int k = threadIdx.x; k < n; k += T) {
                const int e = exact_dist_biased(P[k], P[k + 1]);
                E[k] = (float)e;
                part += e;
            }
            if (threadIdx.x == 0) ls.best[0] = ls.best[1] = 0;
            atomicAdd((unsigned long long*)&ls.len, (unsigned long long)part);
            __syncthreads();
            block_local_search<PACKED>(P, E, tour, n, kNoMoveCap, ls);
            if (ls.len < s_best_len) {  // uniform: ls.len settled before the closing barrier
                for (int k = threadIdx.x; k < n; k += T) best[k] = tour[k];
                __syncthreads();  // everyone has read s_best_len before it changes
                if (threadIdx.x == 0) s_best_len = ls.len;
            }
        }
        if (threadIdx.x == 0 && hist) hist[t + 1] = s_best_len;
        __syncthreads();
    }
    for (int k = threadIdx.x; k < n; k += T) gt[k] = best[k];
    if (threadIdx.x == 0) lengths[b] = s_best_len;
}

size_t batch_smem_bytes(int n) { return (size_t)(n + 1) * (sizeof(float2) + sizeof(float)) + (size_t)n * sizeof(int); }

// + best tour, up to 8 B of alignment, coordinates by city id
size_t batch_ils_smem_bytes(int n)
{
    return batch_smem_bytes(n) + (size_t)n * sizeof(int) + 8 + (size_t)n * sizeof(float2);
}

// Packed windows waste no lanes on short diagonals; per-diagonal windows need
// no wrap logic.  TSP2OPT_BATCH_PACKED=0/1 overrides the size rule.
bool batch_packed(int n)
{
    if (const char* s = getenv("TSP2OPT_BATCH_PACKED")) return atoi(s) != 0;
    return n <= kBatchPackedMaxN;
}

int batch_threads(int n)
{
    if (const char* s = getenv("TSP2OPT_BATCH_THREADS")) {
        const int t = atoi(s);
        if (t >= 32 && t <= kBatchMaxThreads && t % 32 == 0) return t;
    }
    return batch_packed(n) ? 128 : 256;
}

cudaError_t launch_batch_local_search(const int* coords, int* tours, int n, int batch, long long max_iters,
                                      long long* lengths, long long* iters, cudaStream_t st)
{
    const size_t smem = batch_smem_bytes(n);
    const bool packed = batch_packed(n);
    auto kern = packed ? batch_ls_kernel<true> : batch_ls_kernel<false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    kern<<<batch, batch_threads(n), smem, st>>>(coords, tours, n, max_iters, lengths, iters);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_batch_ils(const int* coords, int* tours, int n, int batch, long long iterations,
                             const unsigned long long* seeds, long long* lengths, long long* history, cudaStream_t st)
{
    const size_t smem = batch_ils_smem_bytes(n);
    const bool packed = batch_packed(n);
    auto kern = packed ? batch_ils_kernel<true> : batch_ils_kernel<false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    kern<<<batch, batch_threads(n), smem, st>>>(coords, tours, n, iterations, seeds, lengths, history);
    count_launch();
    return cudaGetLastError();
}

}  // namespace tsp2opt
