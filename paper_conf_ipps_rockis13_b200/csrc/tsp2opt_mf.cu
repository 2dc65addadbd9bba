// tsp2opt_mf.cu -- Multiple Fragment (greedy) start tour on the device
// (L22 §V "an initial solution based on the Multiple
// Fragment(Greedy) heuristic[18]"; definition and tie-break: DESIGN.md R17).
//
// The sequential definition takes edges in increasing key (d, min id, max id)
// and keeps an edge iff both ends have degree < 2 and it closes no cycle.  The
// device reaches the SAME edge set in rounds:
//   * a fragment is a path of kept edges (a single city is a fragment);
//   * an edge is admissible iff it joins ends of two different fragments --
//     once inadmissible, always inadmissible (degrees and fragments only grow);
//   * per round, every fragment end finds its least admissible edge (first
//     admissible entry of its exact K-nearest list, else a scan over all ends);
//     an edge is kept iff it is the least admissible edge of BOTH fragments it
//     joins.  Any smaller edge touching either fragment is inadmissible now and
//     forever, and nothing else can join the two fragments first, so the
//     sequential greedy keeps it too; the globally least admissible edge always
//     qualifies, so every round makes progress.
// The n-1 kept edges form a Hamiltonian path; the closing edge joins its ends.
// The tour (start 0, then 0's lower-id neighbour) is ranked out of the cycle by
// pointer jumping over the 2n directed arcs.
#include "tsp2opt_device.cuh"
#include "tsp2opt_internal.h"

namespace tsp2opt {

namespace {

constexpr unsigned long long kNoEdge = ~0ull;

__device__ __forceinline__ unsigned long long edge_key(int d, int u, int v)
{
    const int a = min(u, v), b = max(u, v);
    return (unsigned long long)d << 44 | (unsigned long long)a << 22 | (unsigned long long)b;
}
__device__ __forceinline__ int edge_other(unsigned long long k, int u)
{
    const int a = (int)(k >> 22 & 0x3FFFFF), b = (int)(k & 0x3FFFFF);
    return a == u ? b : a;
}

// Exact K nearest neighbours of every city by (d, id): brute force over smem
// tiles of coordinates; the squared test s <= dK^2 + dK is exact for
// nint(sqrt(s)) <= dK, so only candidates reach the sqrt.
constexpr int kKnnThreads = 128, kKnnTile = 2048;

__global__ void __launch_bounds__(kKnnThreads) knn_kernel(const int* __restrict__ coords, int n,
                                                          unsigned long long* __restrict__ knn)
{
    __shared__ int2 tile[kKnnTile];
    const int u = blockIdx.x * blockDim.x + threadIdx.x;
    int ux = 0, uy = 0;
    if (u < n) {
        ux = coords[2 * u];
        uy = coords[2 * u + 1];
    }
    unsigned long long key[kMfK];
#pragma unroll
    for (int t = 0; t < kMfK; t++) key[t] = kNoEdge;
    int thr = 0x7FFFFFFF;  // s threshold of the current K-th entry (dK^2 + dK < 2^31)
    for (int base = 0; base < n; base += kKnnTile) {
        const int cnt = min(kKnnTile, n - base);
        __syncthreads();
        for (int t = threadIdx.x; t < cnt; t += blockDim.x)
            tile[t] = make_int2(coords[2 * (base + t)], coords[2 * (base + t) + 1]);
        __syncthreads();
        if (u >= n) continue;
        for (int t = 0; t < cnt; t++) {
            const int2 c = tile[t];
            const int dx = c.x - ux, dy = c.y - uy;
            const int s = dx * dx + dy * dy;
            if (s <= thr && base + t != u) {
                const int d = nint_sqrt_exact(s);
                const unsigned long long k = (unsigned long long)d << 22 | (unsigned long long)(base + t);
                if (k < key[kMfK - 1]) {
                    key[kMfK - 1] = k;
#pragma unroll
                    for (int q = kMfK - 1; q > 0; q--)
                        if (key[q] < key[q - 1]) {
                            const unsigned long long x = key[q];
                            key[q] = key[q - 1];
                            key[q - 1] = x;
                        }
                    if (key[kMfK - 1] != kNoEdge) {
                        const int dk = (int)(key[kMfK - 1] >> 22);
                        thr = dk * dk + dk;
                    }
                }
            }
        }
    }
    if (u < n)
#pragma unroll
        for (int t = 0; t < kMfK; t++) knn[(long long)u * kMfK + t] = key[t];
}

__global__ void mf_init_kernel(int n, int* deg, int* other, int* ptr)
{
    const int u = blockIdx.x * blockDim.x + threadIdx.x;
    if (u < n) {
        deg[u] = 0;
        other[u] = u;
        ptr[u] = 0;
    }
}

// Round phase 1: each fragment end's least admissible edge from its K-list, or
// a request for a full scan.  ctr[par]: [0] ends, [1] scans, [2] accepted,
// [3] kept edges (cumulative, in ctr[kMfEdges]).
__global__ void mf_best_kernel(int n, const unsigned long long* __restrict__ knn, const int* __restrict__ deg,
                               const int* __restrict__ other, int* ptr, unsigned long long* best, int* ends,
                               int* scan, int* ctr, int par)
{
    if (ctr[kMfEdges] >= n - 1) return;
    int* c = ctr + kMfCtr * par;
    const int u = blockIdx.x * blockDim.x + threadIdx.x;
    if (u >= n || deg[u] >= 2) return;
    ends[atomicAdd(&c[0], 1)] = u;
    const int ou = other[u];
    int t = ptr[u];
    unsigned long long b = kNoEdge;
    for (; t < kMfK; t++) {
        const unsigned long long k = knn[(long long)u * kMfK + t];
        if (k == kNoEdge) {
            t = kMfK;
            break;
        }
        const int v = (int)(k & 0x3FFFFF);
        if (deg[v] < 2 && v != ou) {  // admissible
            b = edge_key((int)(k >> 22), u, v);
            break;
        }
    }
    ptr[u] = t;  // entries before t are inadmissible for good
    best[u] = b;
    if (b == kNoEdge) scan[atomicAdd(&c[1], 1)] = u;
}

// Round phase 2: full scans -- one warp per (requesting end, chunk of 1024 ends).
__global__ void mf_scan_kernel(int n, const int* __restrict__ coords, const int* __restrict__ other,
                               unsigned long long* best, const int* __restrict__ ends, const int* __restrict__ scan,
                               const int* ctr, int par)
{
    if (ctr[kMfEdges] >= n - 1) return;
    const int* c = ctr + kMfCtr * par;
    const int ne = c[0], ns = c[1];
    const int chunks = (ne + 1023) / 1024;
    const long long items = (long long)ns * chunks;
    const int lane = threadIdx.x & 31;
    const long long warp0 = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long it = warp0; it < items; it += nwarps) {
        const int u = scan[it / chunks];
        const int ch = (int)(it % chunks);
        const int ou = other[u], ux = coords[2 * u], uy = coords[2 * u + 1];
        unsigned long long b = kNoEdge;
        for (int q = ch * 1024 + lane; q < min(ne, ch * 1024 + 1024); q += 32) {
            const int v = ends[q];
            if (v == u || v == ou) continue;
            const int d = exact_dist_xy(ux, uy, coords[2 * v], coords[2 * v + 1]);
            const unsigned long long k = edge_key(d, u, v);
            b = k < b ? k : b;
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            const unsigned long long x = __shfl_xor_sync(0xffffffffu, b, o);
            b = x < b ? x : b;
        }
        if (lane == 0 && b != kNoEdge) atomicMin(&best[u], b);
    }
}

// Round phase 3: keep an edge iff it is the least admissible edge of both
// fragments it joins (the lower end records it).
__global__ void mf_accept_kernel(int n, const int* __restrict__ other, const unsigned long long* __restrict__ best,
                                 const int* __restrict__ ends, int2* acc, int* ctr, int par)
{
    if (ctr[kMfEdges] >= n - 1) return;
    int* c = ctr + kMfCtr * par;
    const int q = blockIdx.x * blockDim.x + threadIdx.x;
    if (q >= c[0]) return;
    const int u = ends[q];
    const unsigned long long e = best[u];
    if (e == kNoEdge || min(e, best[other[u]]) != e) return;
    const int v = edge_other(e, u);
    if (u > v || min(best[v], best[other[v]]) != e) return;
    acc[atomicAdd(&c[2], 1)] = make_int2(u, v);
}

// Round phase 4: join the accepted fragment pairs (pairwise disjoint, so no
// two accepted edges touch the same fragment); clear the next round's counters.
__global__ void mf_apply_kernel(int n, int* deg, int* other, int* adj, const int2* __restrict__ acc, int* ctr,
                                int par)
{
    int* c = ctr + kMfCtr * par;
    const int q = blockIdx.x * blockDim.x + threadIdx.x;
    if (q == 0) {
        int* nx = ctr + kMfCtr * (par ^ 1);
        nx[0] = nx[1] = nx[2] = 0;
    }
    if (ctr[kMfEdges] >= n - 1 || q >= c[2]) return;
    const int2 e = acc[q];
    const int a = other[e.x], b = other[e.y];
    adj[2 * e.x + deg[e.x]++] = e.y;
    adj[2 * e.y + deg[e.y]++] = e.x;
    other[a] = b;
    other[b] = a;
    atomicAdd(&ctr[kMfEdges], 1);
}

// Close the Hamiltonian path: its ends are the two cities of degree < 2.
__global__ void mf_close_kernel(int n, const int* __restrict__ deg, int* ctr)
{
    const int u = blockIdx.x * blockDim.x + threadIdx.x;
    if (u < n && deg[u] < 2) ctr[kMfEnd0 + (atomicAdd(&ctr[kMfEndCnt], 1) & 1)] = u;
}

__global__ void mf_close2_kernel(int* deg, int* adj, const int* ctr)
{
    const int a = ctr[kMfEnd0], b = ctr[kMfEnd0 + 1];
    adj[2 * a + deg[a]++] = b;
    adj[2 * b + deg[b]++] = a;
}

// Tour ranking over directed arcs a = 2u + s (u -> adj[a]); succ(a) leaves
// v = adj[a] through the slot not pointing back to u.  The arc into city 0
// that precedes the start arc (0 -> lower-id neighbour) is cut, so the start
// arc's cycle becomes a list; Wyllie pointer jumping ranks it.
__global__ void arc_init_kernel(int n, const int* __restrict__ adj, int* nxt, int* rank)
{
    const int a = blockIdx.x * blockDim.x + threadIdx.x;
    if (a >= 2 * n) return;
    const int u = a >> 1, v = adj[a];
    int s = (adj[2 * v] == u) ? 1 : 0;
    int succ = 2 * v + s;
    // cut: the arc w -> 0 whose successor is the start arc
    const int s0 = adj[0] < adj[1] ? 0 : 1;  // start arc: 0 -> its lower-id neighbour
    if (v == 0 && succ == s0) succ = -1;
    nxt[a] = succ;
    rank[a] = succ < 0 ? 0 : 1;
}

__global__ void arc_jump_kernel(int n, const int* __restrict__ nxt_in, const int* __restrict__ rank_in, int* nxt_out,
                                int* rank_out)
{
    const int a = blockIdx.x * blockDim.x + threadIdx.x;
    if (a >= 2 * n) return;
    const int s = nxt_in[a];
    if (s < 0) {
        nxt_out[a] = -1;
        rank_out[a] = rank_in[a];
    } else {
        nxt_out[a] = nxt_in[s];
        rank_out[a] = rank_in[a] + rank_in[s];
    }
}

__global__ void arc_scatter_kernel(int n, const int* __restrict__ nxt, const int* __restrict__ rank, int* tour)
{
    const int a = blockIdx.x * blockDim.x + threadIdx.x;
    if (a >= 2 * n || nxt[a] >= 0) return;  // arcs of the reversed cycle never reach the cut
    tour[n - 1 - rank[a]] = a >> 1;
}

inline int blocks(long long work, int t) { return (int)((work + t - 1) / t); }

}  // namespace

// Workspace layout (one allocation per handle, reused by every call).
struct MfLayout {
    size_t off[15];
    size_t total;
    explicit MfLayout(int n)
    {
        const size_t N = (size_t)n;
        const size_t sz[15] = {N * kMfK * 8, N * 8, N * 4, N * 4, N * 4, N * 4, N * 4,
                               N * 8,        N * 8, N * 8, N * 8, N * 8, N * 8, kMfCtrInts * 4, 0};
        total = 0;
        for (int k = 0; k < 15; k++) {
            off[k] = total;
            total += (sz[k] + 255) / 256 * 256;
        }
    }
};

size_t mf_workspace_bytes(int n) { return MfLayout(n).total; }

cudaError_t launch_knn(const int* coords, int n, unsigned long long* knn, cudaStream_t st)
{
    knn_kernel<<<blocks(n, kKnnThreads), kKnnThreads, 0, st>>>(coords, n, knn);
    count_launch(1);
    return cudaGetLastError();
}

cudaError_t launch_mf_tour(const int* coords, int n, void* ws, int* tour_out, int* rounds_out, cudaStream_t st)
{
    const MfLayout L(n);
    char* p = static_cast<char*>(ws);
    const size_t N = (size_t)n;
    auto* knn = reinterpret_cast<unsigned long long*>(p + L.off[0]);
    auto* best = reinterpret_cast<unsigned long long*>(p + L.off[1]);
    int* deg = reinterpret_cast<int*>(p + L.off[2]);
    int* other = reinterpret_cast<int*>(p + L.off[3]);
    int* ptr = reinterpret_cast<int*>(p + L.off[4]);
    int* ends = reinterpret_cast<int*>(p + L.off[5]);
    int* scan = reinterpret_cast<int*>(p + L.off[6]);
    auto* acc = reinterpret_cast<int2*>(p + L.off[7]);
    int* adj = reinterpret_cast<int*>(p + L.off[8]);
    int* nxt0 = reinterpret_cast<int*>(p + L.off[9]);
    int* rk0 = reinterpret_cast<int*>(p + L.off[10]);
    int* nxt1 = reinterpret_cast<int*>(p + L.off[11]);
    int* rk1 = reinterpret_cast<int*>(p + L.off[12]);
    int* ctr = reinterpret_cast<int*>(p + L.off[13]);
    cudaError_t e;
    if ((e = cudaMemsetAsync(ctr, 0, kMfCtrInts * 4, st)) != cudaSuccess) return e;
    knn_kernel<<<blocks(n, kKnnThreads), kKnnThreads, 0, st>>>(coords, n, knn);
    mf_init_kernel<<<blocks(n, 256), 256, 0, st>>>(n, deg, other, ptr);
    count_launch(2);
    // rounds, checked for completion in batches (extra rounds exit at once)
    int rounds = 0, h_edges = 0;
    int* h_ctr = nullptr;
    if ((e = cudaMallocHost(&h_ctr, kMfCtrInts * 4)) != cudaSuccess) return e;
    const int scan_grid = 148 * 8;
    for (int batch = 4; h_edges < n - 1; batch = min(batch * 2, 16)) {
        for (int r = 0; r < batch; r++, rounds++) {
            const int par = rounds & 1;
            mf_best_kernel<<<blocks(n, 256), 256, 0, st>>>(n, knn, deg, other, ptr, best, ends, scan, ctr, par);
            mf_scan_kernel<<<scan_grid, 256, 0, st>>>(n, coords, other, best, ends, scan, ctr, par);
            mf_accept_kernel<<<blocks(n, 256), 256, 0, st>>>(n, other, best, ends, acc, ctr, par);
            mf_apply_kernel<<<blocks(n, 256), 256, 0, st>>>(n, deg, other, adj, acc, ctr, par);
            count_launch(4);
        }
        if ((e = cudaMemcpyAsync(h_ctr, ctr, kMfCtrInts * 4, cudaMemcpyDeviceToHost, st)) != cudaSuccess) break;
        if ((e = cudaStreamSynchronize(st)) != cudaSuccess) break;
        if ((e = cudaGetLastError()) != cudaSuccess) break;
        h_edges = h_ctr[kMfEdges];
        if (rounds > 4 * n + 64) {  // cannot happen: every round keeps >= 1 edge
            e = cudaErrorUnknown;
            break;
        }
    }
    cudaFreeHost(h_ctr);
    if (e != cudaSuccess) return e;
    mf_close_kernel<<<blocks(n, 256), 256, 0, st>>>(n, deg, ctr);
    mf_close2_kernel<<<1, 1, 0, st>>>(deg, adj, ctr);
    arc_init_kernel<<<blocks(2 * N, 256), 256, 0, st>>>(n, adj, nxt0, rk0);
    count_launch(3);
    int steps = 1;
    while ((1LL << steps) < 2LL * n) steps++;
    for (int s = 0; s < steps; s++) {
        arc_jump_kernel<<<blocks(2 * N, 256), 256, 0, st>>>(n, nxt0, rk0, nxt1, rk1);
        std::swap(nxt0, nxt1);
        std::swap(rk0, rk1);
    }
    arc_scatter_kernel<<<blocks(2 * N, 256), 256, 0, st>>>(n, nxt0, rk0, tour_out);
    count_launch(steps + 1);
    if (rounds_out) *rounds_out = rounds;
    return cudaGetLastError();
}

}  // namespace tsp2opt
