// tsp2opt_device.cuh -- device-side arithmetic of the sm_100a 2-opt path.
//
// Shared by the sweep, apply, load and self-test kernels of libtsp2opt.so only
// (never by oracle/).  Citations: PAPER.md line = page;
// readings R1..R13 in DESIGN.md §3.
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace tsp2opt {

// ---------------------------------------------------------------------------
// Packed best-move key (reading R5: lowest delta, then lowest Fig. 3 cell
// k = j(j-1)/2 + i, i.e. lowest j then lowest i):
//   key = (delta + 2^18) << 44 | j << 22 | i,  bit 63 == 0,
// so unsigned and signed int64 order agree (atomicMin(u64), NCCL MIN on int64).
// |delta| <= 2 * 46340 < 2^18 and n <= 2^22.
// ---------------------------------------------------------------------------
constexpr int kKeyDeltaShift = 44;
constexpr int kKeyJShift = 22;
constexpr int kDeltaBias = 1 << 18;
constexpr unsigned long long kKeyNone = ~0ULL;

// sweep option bits (tsp2opt_set_option)
constexpr int kSweepSeed = 1;        // seed each tile with its surviving minimum of the previous sweep
constexpr int kSweepTileBounds = 2;  // skip tiles whose bounding boxes prove that no pair passes the filter
constexpr int kSweepLocal = 4;       // tile-local bound (start at delta < 0, ignore the global key): the tile's
                                     // minimum is then exact on its own and can be reused while the tile is clean
constexpr int kSweepIncremental = 8; // culled sweep: only tiles the last applied move touched are re-swept
constexpr int kSweepFull = 16;       // incremental sweep whose stored minima are not valid yet: re-sweep all
// First improvement (reading R20): improving pairs enter the min with this
// delta, so the min is the lowest cell; first_fix_kernel writes the real delta.
constexpr int kFirstDelta = -1;
constexpr int kSweepFirst = 32;      // first improvement: the lowest improving cell instead of the lowest delta
constexpr int kSweepPartBounds = 64; // inc_ls2: the bounding-box test of tile_may_pass on each column part

// Bounding box of a run of route positions (unbiased integer coordinates) and
// the largest tour edge leaving it: the summaries the tile cull compares.
struct __align__(32) Box {
    int xlo, xhi, ylo, yhi;
    int emax;
    int pad[3];
};

__host__ __device__ __forceinline__ unsigned long long pack_key(int delta, int i, int j)
{
    return ((unsigned long long)(unsigned)(delta + kDeltaBias) << kKeyDeltaShift) |
           ((unsigned long long)(unsigned)j << kKeyJShift) | (unsigned long long)(unsigned)i;
}
__host__ __device__ __forceinline__ int key_delta(unsigned long long k)
{
    return (int)(k >> kKeyDeltaShift) - kDeltaBias;
}
__host__ __device__ __forceinline__ int key_j(unsigned long long k) { return (int)((k >> kKeyJShift) & 0x3FFFFF); }
__host__ __device__ __forceinline__ int key_i(unsigned long long k) { return (int)(k & 0x3FFFFF); }

// The degenerate pair (0,1) has delta 0 and cell 0 (reading R7): every sweep
// starts from it, so a sweep at a local minimum returns (0, 1, 0).
__host__ __device__ __forceinline__ unsigned long long seed_key() { return pack_key(0, 0, 1); }

// ---------------------------------------------------------------------------
// Coordinates live on the device as float(x + 2^23): the float difference of
// two such values is the exact integer difference (same exponent, ulp 1), and
// the raw bits minus 0x4B000000 give x back for the exact integer path.
// ---------------------------------------------------------------------------
constexpr float kCoordBias = 8388608.0f;  // 2^23
__host__ __device__ __forceinline__ float bias_coord(int x) { return (float)(x + (1 << 23)); }
__device__ __forceinline__ int unbias(float f) { return __float_as_int(f) - 0x4B000000; }

// Programmatic dependent launch (sm_90+): a kernel launched with the PDL
// attribute may be dispatched while its predecessor drains; pdl_wait() blocks
// until the predecessor grid has completed and its writes are visible (a no-op
// without the attribute), pdl_trigger() lets the successor be dispatched.  The
// iteration kernels call both first thing, before any global access, so the
// only overlap is launch latency and CTA dispatch -- never data.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

__device__ __forceinline__ float sqrt_approx(float x)
{
    float r;
    asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
    return r;
}

// Exact TSPLIB EUC_2D nint(sqrt(s)) for 0 <= s <= 2*32767^2 (reading R3/R4):
// one MUFU.SQRT estimate rounded to the nearest integer m, then one integer
// correction step using  nint(sqrt(s)) = m  <=>  m^2 - m < s <= m^2 + m.
// Exhaustively verified on the device over every s (tsp2opt_selftest).
__device__ __forceinline__ int nint_sqrt_exact(int s)
{
    float r = sqrt_approx(__int2float_rn(s));
    int m = __float2int_rn(r);
    long long ss = s, mm = (long long)m * m;
    if (ss > mm + m) m += 1;
    else if (m > 0 && ss <= mm - m) m -= 1;  // m = 0: nothing is below 0
    return m;
}

// nint(sqrt(s)) from the float squared distance s_f = fma(dx, dx, dy*dy) of
// exact dx, dy, when the float path is unambiguous: |sqrt_approx(s_f) - sqrt(s)|
// < 0.03 (MUFU.SQRT relative error <= 2^-21, tsp2opt_selftest_sqrt; s_f within
// 2^-23 of s), so a nearest integer m with |sqrt_approx(s_f) - m| < 0.45 is
// nint(sqrt(s)).  Returns false (out untouched) otherwise.  Exhaustively
// checked over every (dx, dy) by tsp2opt_selftest.
__device__ __forceinline__ bool nint_from_float(float s_f, float& out)
{
    const float r = sqrt_approx(s_f);
    const float m = (r + 12582912.0f) - 12582912.0f;  // 1.5 * 2^23: nearest integer (exact)
    if (fabsf(r - m) < 0.45f) {
        out = m;
        return true;
    }
    return false;
}

__device__ __forceinline__ int exact_dist_xy(int xa, int ya, int xb, int yb)
{
    int dx = xa - xb, dy = ya - yb;
    return nint_sqrt_exact(dx * dx + dy * dy);
}

__device__ __forceinline__ int exact_dist_biased(float2 a, float2 b)
{
    return exact_dist_xy(unbias(a.x), unbias(a.y), unbias(b.x), unbias(b.y));
}

// ---------------------------------------------------------------------------
// Squared-distance prefilter.  For an integer t:
//   nint(sqrt(s)) <= t  <=>  s <= t^2 + t   (t >= 0; impossible for t < 0).
// sq_threshold(t) returns a float S_f >= (t^2 + t)(1 + 2^-21) for t >= 0 and a
// negative value for t < 0.  The float squared distance s_f = fma(dx,dx,dy*dy)
// satisfies s_f <= s (1 + 2^-23 + 2^-48) (two roundings, exact dx, dy), so
// s <= t^2 + t  implies  s_f <= S_f: the filter never rejects a pair the exact
// test would accept.  Exhaustively verified on the device (tsp2opt_selftest).
// ---------------------------------------------------------------------------
constexpr float kThrScale = 1.00000095367431640625f;  // 1 + 2^-20
__device__ __forceinline__ float sq_threshold(float t)
{
    float tt = fmaxf(t, -0.5f);            // t < 0  ->  tt^2 + tt = -0.25 < 0
    return fmaf(tt, tt, tt) * kThrScale;
}

// ---------------------------------------------------------------------------
// Blackwell packed FP32x2 arithmetic (FADD2 / FMUL2 / FFMA2): one issue slot
// for two lanes' worth of FP32 work.
// ---------------------------------------------------------------------------
__device__ __forceinline__ float2 add2(float2 a, float2 b)
{
    float2 r;
    asm("{\n\t.reg .b64 ra, rb, rd;\n\t"
        "mov.b64 ra, {%2, %3};\n\tmov.b64 rb, {%4, %5};\n\t"
        "add.rn.f32x2 rd, ra, rb;\n\tmov.b64 {%0, %1}, rd;\n\t}"
        : "=f"(r.x), "=f"(r.y) : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y));
    return r;
}
__device__ __forceinline__ float2 mul2(float2 a, float2 b)
{
    float2 r;
    asm("{\n\t.reg .b64 ra, rb, rd;\n\t"
        "mov.b64 ra, {%2, %3};\n\tmov.b64 rb, {%4, %5};\n\t"
        "mul.rn.f32x2 rd, ra, rb;\n\tmov.b64 {%0, %1}, rd;\n\t}"
        : "=f"(r.x), "=f"(r.y) : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y));
    return r;
}
__device__ __forceinline__ float2 fma2(float2 a, float2 b, float2 c)
{
    float2 r;
    asm("{\n\t.reg .b64 ra, rb, rc, rd;\n\t"
        "mov.b64 ra, {%2, %3};\n\tmov.b64 rb, {%4, %5};\n\tmov.b64 rc, {%6, %7};\n\t"
        "fma.rn.f32x2 rd, ra, rb, rc;\n\tmov.b64 {%0, %1}, rd;\n\t}"
        : "=f"(r.x), "=f"(r.y)
        : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y), "f"(c.x), "f"(c.y));
    return r;
}

// min over v[LO..HI) as a balanced tree of 3-input minima (FMNMX3): depth
// log3 instead of the linear chain a fold would produce.
template <int LO, int HI>
__device__ __forceinline__ float tree_min(const float* v)
{
    static_assert(HI > LO, "empty range");
    if constexpr (HI - LO == 1) {
        return v[LO];
    } else if constexpr (HI - LO == 2) {
        return fminf(v[LO], v[LO + 1]);
    } else if constexpr (HI - LO == 3) {
        return fminf(fminf(v[LO], v[LO + 1]), v[LO + 2]);
    } else {
        constexpr int M1 = LO + (HI - LO) / 3, M2 = LO + 2 * (HI - LO) / 3;
        return fminf(fminf(tree_min<LO, M1>(v), tree_min<M1, M2>(v)), tree_min<M2, HI>(v));
    }
}

// 32-bit shared-memory addressing (keeps the fast loop free of generic->shared
// conversions).
__device__ __forceinline__ unsigned smem_addr(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ float4 lds4(unsigned a)
{
    float4 v;
    asm("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(a));
    return v;
}
__device__ __forceinline__ float2 lds2(unsigned a)
{
    float2 v;
    asm("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(v.x), "=f"(v.y) : "r"(a));
    return v;
}

// Squared distances of two row cities (packed) to one column city given as
// negated biased coordinates (-x, -x) / (-y, -y):  s = dx*dx + dy*dy.
__device__ __forceinline__ float2 sq2(float2 xr, float2 yr, float2 ncx, float2 ncy)
{
#ifdef TSP2OPT_SCALAR_SQ  // experiment: scalar FADD/FMUL/FFMA instead of the packed FP32x2 forms
    const float dx0 = xr.x + ncx.x, dx1 = xr.y + ncx.y, dy0 = yr.x + ncy.x, dy1 = yr.y + ncy.y;
    return make_float2(fmaf(dx0, dx0, dy0 * dy0), fmaf(dx1, dx1, dy1 * dy1));
#else
    float2 dx = add2(xr, ncx);
    float2 dy = add2(yr, ncy);
    return fma2(dx, dx, mul2(dy, dy));
#endif
}

// ILS perturbation cuts (reading R16; L18 §V "a simple doublebridge move"):
// splitmix64 output 3*it + k of `seed` gives the k-th segment length
// 1 + out % max(1, (n-1)/3); a = l0, b = a + l1, c = b + l2
// (1 <= a < b < c <= n-1).  Used on the host (tsp2opt_ils) and on the device
// (batched ILS); the oracle implements the same counter-based generator on
// its own.
__host__ __device__ __forceinline__ uint64_t splitmix64_at(uint64_t seed, uint64_t k)
{
    uint64_t z = seed + (k + 1) * 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

__host__ __device__ __forceinline__ void ils_cuts(long long n, uint64_t seed, long long it, long long* a,
                                                  long long* b, long long* c)
{
    const unsigned long long m = (unsigned long long)((n - 1) / 3 > 1 ? (n - 1) / 3 : 1);  // max(1, (n-1)/3)
    const long long l0 = 1 + (long long)(splitmix64_at(seed, 3ULL * it) % m);
    const long long l1 = 1 + (long long)(splitmix64_at(seed, 3ULL * it + 1) % m);
    const long long l2 = 1 + (long long)(splitmix64_at(seed, 3ULL * it + 2) % m);
    *a = l0;
    *b = l0 + l1;
    *c = l0 + l1 + l2;
}

// A pair (a, b) of the tour before the 2-opt move (i, j) -- positions i+1..j
// reversed -- keeps its delta in the new tour iff both its edges lie on the same
// side of the reversed segment: both outside keep their positions, both inside
// move to (i+j-b, i+j-a).  Returns the pair's key in the new tour, or kKeyNone.
// Any such key is a real pair of the new tour with its exact delta, hence a
// valid upper bound on the next sweep's minimum (every pair is still examined).
__host__ __device__ __forceinline__ unsigned long long surviving_key(unsigned long long k, int i, int j)
{
    if (k == kKeyNone) return kKeyNone;
    const int a = key_i(k), b = key_j(k);
    const bool ain = a >= i + 1 && a <= j - 1, aout = a <= i - 1 || a >= j + 1;
    const bool bin = b >= i + 1 && b <= j - 1, bout = b <= i - 1 || b >= j + 1;
    if (aout && bout) return k;
    if (ain && bin) return pack_key(key_delta(k), i + j - b, i + j - a);
    return kKeyNone;
}

// Per-rank / per-handle device state, ping-ponged between iterations: the
// kernels of iteration t read slot[t & 1] and write slot[(t + 1) & 1], so no
// kernel ever reads a field another block of the same kernel writes.
struct __align__(64) Slot {
    unsigned long long key;       // best-move key of the sweep reading this slot (atomicMin target)
    unsigned long long last_key;  // key of the most recent finished sweep
    long long moves;              // moves applied since the tour was loaded
    long long length;             // current tour length (int64: n * 46340 > 2^31)
    int done;                     // 0 running, 1 local minimum, 2 capped, bit 2 (4): invalid tour,
                                  // bit 3 (8): peer exchange timed out
    unsigned next_tile;           // culled sweep: next entry of the kept-tile list to claim
    int seed_ok;                  // 1: last_key is the move just applied to the tour the tile minima of the
                                  //    previous sweep were measured on (they may seed this sweep)
    unsigned ncull;               // culled sweep: number of kept tiles in the list
    int mtype;                    // 2.5-opt: type of the move last applied / decided (reading R19)
    int pad[3];
};

// Slot::done bit set when a peer-memory exchange timed out (tsp2opt_p2p.cu).
constexpr int kDoneExchangeTimeout = 8;

// Peer-memory exchange of the per-sweep key (tsp2opt_p2p.cu): written by the
// peers, polled by the owner; [parity][source rank].
constexpr int kP2PMaxWorld = 8;
struct __align__(64) Mailbox {
    unsigned long long key[2][kP2PMaxWorld];
    unsigned long long seq[2][kP2PMaxWorld];
    unsigned long long counter;  // exchanges completed by the owner
};

// Software grid barrier for co-resident grids (cooperative launches): arrive
// on bar[0], the last block resets it and advances the generation bar[1].
__device__ __forceinline__ void grid_sync(unsigned* bar, unsigned nblocks)
{
    __syncthreads();
    if (threadIdx.x == 0) {
        volatile unsigned* vgen = bar + 1;
        const unsigned gen = *vgen;
        __threadfence();
        if (atomicAdd(bar, 1u) == nblocks - 1) {
            atomicExch(bar, 0u);
            __threadfence();
            atomicAdd(bar + 1, 1u);
        } else {
            while (*vgen == gen) __nanosleep(32);  // (a busy spin measured the same, r02)
        }
        __threadfence();
    }
    __syncthreads();
}

#ifndef TSP2OPT_BAR_ACQREL
#define TSP2OPT_BAR_ACQREL 1  // measured 2 % faster per move than two __threadfence()s (MEMBAR.ALL vs .SC)
#endif
// Grid barrier on a monotonic 64-bit arrival counter (reset to 0 before the
// launch; every barrier of the launch adds gridDim.x): one atomic per CTA and
// polling, no reset round trips.  `target` is the CTA's running count.
__device__ __forceinline__ void grid_sync_mono(unsigned long long* ctr, unsigned long long& target)
{
    __syncthreads();
    target += gridDim.x;
    if (threadIdx.x == 0) {
#if TSP2OPT_BAR_ACQREL
        // release-add / acquire-poll at gpu scope instead of two full fences
        asm volatile("red.release.gpu.global.add.u64 [%0], 1;" ::"l"(ctr) : "memory");
        unsigned long long v;
        do {
            asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(ctr) : "memory");
        } while (v < target);
#else
        __threadfence();
        atomicAdd(ctr, 1ULL);
        while (*(volatile unsigned long long*)ctr < target) {
        }
        __threadfence();
#endif
    }
    __syncthreads();
}

// Grid barrier on a monotonic 64-bit counter that is never reset: the arrival's
// old value gives the generation (every launch on the counter uses the same grid
// and passes every barrier, so the counter is a multiple of the grid between
// launches).  Release-add / acquire-poll at gpu scope, as grid_sync_mono.
__device__ __forceinline__ void grid_sync_gen(unsigned long long* ctr)
{
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long old;
        asm volatile("atom.release.gpu.global.add.u64 %0, [%1], 1;" : "=l"(old) : "l"(ctr) : "memory");
        const unsigned long long target = (old / gridDim.x + 1) * gridDim.x;
        unsigned long long v;
        do {
            asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(ctr) : "memory");
        } while (v < target);
    }
    __syncthreads();
}

}  // namespace tsp2opt
