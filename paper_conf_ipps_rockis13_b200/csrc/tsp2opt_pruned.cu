// tsp2opt_pruned.cu -- neighbourhood-pruned best-improvement 2-opt sweep
// (SURVEY.md §8(f) NEXT-4).  L18 §V: "Possibly limiting the neighborhood
// would also bring an improvement in efficiency"; L26 §VII: "simple ideas such
// as neighborhood pruning can be applied at the cost of the quality of the
// solution".  Reading R18 fixes the K-nearest-neighbour rule:
//   N_K(a) = the K cities c != a with the smallest (d(a,c), c),
//   E_K    = { {a,c} : c in N_K(a) or a in N_K(c) },
//   M_K    = the 2-opt pairs (i, j) of the closed tour whose move creates an
//            edge of E_K: {t[i], t[j]} or {t[i+1], t[j+1]} in E_K.
// The best move is the lowest (delta, Fig. 3 cell) over M_K with delta < 0,
// else the seed (0, 1, 0) -- the same packed key and tie-break as the full
// sweep (reading R5), so the result is bit-exact with oracle_pruned_best_move.
//
// Enumeration: with p, q the positions of a and c (a candidate edge c in
// N_K(a)) and prev(x) = (x - 1) mod n, the two moves creating {a, c} are
//   sorted(p, q)              {t[i], t[j]} = {a, c}:
//       delta = d(a,c) + D(P[p+1], P[q+1]) - E[p] - E[q]
//   sorted(prev p, prev q)    {t[i+1], t[j+1]} = {a, c} (position 0 is
//                             position n of the closed tour, so u = 0 gives
//                             (v-1, n-1)):
//       delta = d(a,c) + D(P[prev p], P[prev q]) - E[prev p] - E[prev q]
// Every pair of M_K is reached this way (from either end of its candidate
// edge), and nothing else is.  d(a, c) comes from the exact K-NN key; the
// other new edge is computed exactly (float path when unambiguous, else the
// integer nint).  Work per sweep: n K candidates, 2 moves
// each -- O(nK) instead of C(n,2).
//
// One thread owns 1/TP of the candidate list of one position: its own
// P[p+1], P[prev p], E[p], E[prev p] are coalesced loads, its candidates'
// pos[c] and then P / E around q are independent gathers, all issued before
// any is used.  The dependent chain tour -> knn -> pos -> P/E makes the sweep
// L2-latency bound; pos is kept current by the apply kernel.
#include "tsp2opt_device.cuh"
#include "tsp2opt_internal.h"

#include <cstdlib>

namespace tsp2opt {

namespace {

constexpr int kPrunedThreads = 128;

__device__ __forceinline__ int exact_edge(float2 a, float2 b)
{
    const float dx = a.x - b.x, dy = a.y - b.y;  // exact: biased floats share the exponent
    float d;
    if (nint_from_float(fmaf(dx, dx, dy * dy), d)) return (int)d;
    return exact_dist_biased(a, b);
}

__device__ __forceinline__ unsigned long long umin64(unsigned long long a, unsigned long long b) { return a < b ? a : b; }

// Key of the move (i, j) = sorted(x, y) whose other new edge joins ax and ay;
// dn is the exact length of the candidate edge, ex and ey the two removed edges.
// delta >= dn - ex - ey (the other new edge is >= 0): no sqrt when that is >= 0.
// first != 0 (first improvement, reading R20): improving moves enter the min
// with the marker delta kFirstDelta, so the min is the lowest cell.
__device__ __forceinline__ unsigned long long move_key(int x, int y, float2 ax, float2 ay, int dn, int ex, int ey,
                                                       int first)
{
    const int lo = dn - ex - ey;
    if (lo >= 0) return kKeyNone;
    const int d = lo + exact_edge(ax, ay);
    return d < 0 ? pack_key(first ? kFirstDelta : d, min(x, y), max(x, y)) : kKeyNone;
}

}  // namespace

// a4 + a5 over M_K: candidates of positions [p0, p1) (this rank's share);
// TP threads per position, thread s of a position takes candidates s, s+TP, ...
template <int TP>
__global__ void __launch_bounds__(kPrunedThreads) pruned_sweep_kernel(
    const float2* __restrict__ P, const int* __restrict__ E, const int* __restrict__ tour, const int* __restrict__ pos,
    const unsigned long long* __restrict__ knn, int K, int n, int p0, int p1, Slot* __restrict__ slot,
    int respect_done, int first)
{
    constexpr int kSlots = kMaxNeighbours / TP;
    pdl_trigger();
    pdl_wait();
    if (respect_done && *(volatile int*)&slot->done) return;  // converged: iteration is a no-op
    const int gid = blockIdx.x * blockDim.x + threadIdx.x;
    const int p = p0 + gid / TP, s0 = gid % TP;
    unsigned long long best = kKeyNone;
    if (p < p1) {
        // Threads follow positions, not city ids: consecutive positions of a
        // coherent tour have nearby candidates, so the gathers share lines
        // (measured: by-city order one dependent load shorter but 15-30 %
        // slower at n = 33810 / 85900, profiles/r01_pruned_variants.jsonl).
        const int a = __ldg(tour + p), pa = p;
        const int pp = pa == 0 ? n - 1 : pa - 1;
        const float2 a1 = __ldg(P + pa + 1), a0 = __ldg(P + pp);
        const int ea1 = __ldg(E + pa), ea0 = __ldg(E + pp);
        unsigned long long nk[kSlots];
        int q[kSlots];
#pragma unroll
        for (int r = 0; r < kSlots; r++) {
            const int t = s0 + r * TP;
            nk[r] = t < K ? __ldg(knn + (long long)a * kMaxNeighbours + t) : ~0ull;  // (d << 22 | c), by (d, c)
        }
#pragma unroll
        for (int r = 0; r < kSlots; r++) q[r] = nk[r] != ~0ull ? __ldg(pos + (int)(nk[r] & 0x3FFFFF)) : -1;
#pragma unroll
        for (int r = 0; r < kSlots; r++) {
            if (q[r] < 0) continue;
            const int qq = q[r], qp = qq == 0 ? n - 1 : qq - 1, dac = (int)(nk[r] >> 22);
            const float2 c1 = __ldg(P + qq + 1), c0 = __ldg(P + qp);
            const int ec1 = __ldg(E + qq), ec0 = __ldg(E + qp);
            best = umin64(best, move_key(pa, qq, a1, c1, dac, ea1, ec1, first));  // {t[i], t[j]} = {a, c}
            best = umin64(best, move_key(pp, qp, a0, c0, dac, ea0, ec0, first));  // {t[i+1], t[j+1]} = {a, c}
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) best = umin64(best, __shfl_xor_sync(0xffffffffu, best, o));
    __shared__ unsigned long long s_red[kPrunedThreads / 32];
    if ((threadIdx.x & 31) == 0) s_red[threadIdx.x >> 5] = best;
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long m = s_red[0];
        for (int w = 1; w < kPrunedThreads / 32; w++) m = umin64(m, s_red[w]);
        if (m < *(volatile unsigned long long*)&slot->key) atomicMin(&slot->key, m);
    }
}

// pos[tour[k]] = k: the inverse permutation the enumeration needs (the apply
// kernel keeps it current across reversals).
__global__ void pos_kernel(const int* __restrict__ tour, int* __restrict__ pos, int n)
{
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k < n) pos[tour[k]] = k;
}

static int pruned_tp(int n)
{
    if (const char* e = getenv("TSP2OPT_PRUNED_TP")) {
        const int v = atoi(e);
        if (v == 1 || v == 2 || v == 4 || v == 8) return v;
    }
    return n >= 40000 ? 2 : 4;
}

cudaError_t launch_pruned_sweep(const float2* P, const int* E, const int* tour, const int* pos,
                                const unsigned long long* knn, int K, int n, int p0, int p1, Slot* slot,
                                int respect_done, int first, cudaStream_t st)
{
    const int tp = pruned_tp(n);
    const long long threads = (long long)std::max(0, p1 - p0) * tp;
    const dim3 grid((unsigned)std::max(1LL, (threads + kPrunedThreads - 1) / kPrunedThreads)), block(kPrunedThreads);
    cudaError_t e;
#define TSP2OPT_PRUNED_LAUNCH(T) \
    launch_kernel_pdl(pruned_sweep_kernel<T>, grid, block, 0, st, P, E, tour, pos, knn, K, n, p0, p1, slot, respect_done, \
                      first)
    switch (tp) {
    case 1: e = TSP2OPT_PRUNED_LAUNCH(1); break;
    case 2: e = TSP2OPT_PRUNED_LAUNCH(2); break;
    case 8: e = TSP2OPT_PRUNED_LAUNCH(8); break;
    default: e = TSP2OPT_PRUNED_LAUNCH(4); break;
    }
#undef TSP2OPT_PRUNED_LAUNCH
    if (e != cudaSuccess) return e;
    count_launch(1);
    return cudaGetLastError();
}

cudaError_t launch_pos(const int* tour, int* pos, int n, cudaStream_t st)
{
    pos_kernel<<<(n + 255) / 256, 256, 0, st>>>(tour, pos, n);
    count_launch(1);
    return cudaGetLastError();
}

}  // namespace tsp2opt
