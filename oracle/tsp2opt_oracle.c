/*
 * oracle/tsp2opt_oracle.c -- plain CPU oracle for exhaustive best-improvement
 * 2-opt on the symmetric Euclidean TSP (Rocki & Suda, IPDPSW 2013).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_ipps_rockis13_b200/, libtsp2opt.so) never
 * links, imports or calls it, and this file shares no code, header, table or
 * constant generator with the CUDA path.
 *
 * Everything is int64 integer arithmetic (the paper fixes no float precision
 * for the oracle; distances are TSPLIB EUC_2D on integer coordinates, so every
 * quantity the method computes is an integer and the oracle is exact).
 *
 * Citations: PAPER.md is one physical line per paper page:
 *   L12 = p.2 (§I.B 2-opt, Fig. 1, Fig. 2), L14 = p.3 (§IV, Fig. 3, Alg. 2),
 *   L16 = p.4 (Listing 1, §IV.A), L18 = p.5 (Fig. 6, §IV.B).
 * Readings R1..R13 of garbled / silent passages are listed in DESIGN.md §3.
 *
 * Parity pins (tests/test_oracle.py, tests/test_oracle_dist.py):
 *   oracle_dist       -- closed form nint = (isqrt(4s)+1)//2 (Python, exhaustive
 *                        boundaries), exhaustive C cross-check over all s.
 *   oracle_best_move  -- brute force: every 2-opt neighbour built by explicit
 *                        reversal and full length recomputation, n <= 9;
 *                        Fig. 2 worked example; Fig. 3 cell order.
 *   oracle_apply      -- Fig. 2 worked example; permutation invariant.
 *   oracle_local_search -- delta == full recomputation after every move,
 *                        local-minimum certificate, convex-position hull order,
 *                        brute-force global optimum is a 2-opt local minimum.
 *   oracle_knn, oracle_pruned_* (tests/test_oracle_pruned.py) -- K nearest by
 *                        a Python sort of (nint, id); best pruned move by brute
 *                        force over explicitly built neighbours whose CREATED
 *                        edges (edge-set difference) meet E_K; K >= n-1 equals
 *                        the full oracle; list enumeration == plain scan.
 *   oracle25_* (tests/test_oracle_25opt.py) -- 2.5-opt: brute force over
 *                        neighbours built from the move's wording with list
 *                        operations on city ids; the neighbourhood as a set of
 *                        cycles == 2-opt neighbours + node insertions; the
 *                        sweep == the per-move definition; global optima.
 *   oracleor_* (tests/test_oracle_oropt.py) -- Or-opt (reading R21): brute
 *                        force over neighbours built from the move's wording
 *                        (cut a segment of L cities, insert it after a city);
 *                        the neighbourhood as a set of cycles == 2-opt
 *                        neighbours + all segment moves; L = 1 == 2.5-opt's
 *                        insertions; the optimum admits no improving move.
 *   oracle_first_* (tests/test_oracle_first.py) -- first improvement: the
 *                        first improving neighbour of an explicit scan in cell
 *                        order; 2-opt local-minimum certificate.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* ---------------------------------------------------------------------------
 * Distance.  L16 Listing 1: "return (int)(sqrtf(dx*dx+dy*dy) + 0.5f); //
 * return Euclidean distance" -- the intent is the TSPLIB EUC_2D rounded
 * Euclidean distance nint(sqrt(dx^2+dy^2)).  Reading R3: we compute that
 * integer exactly (Listing 1's float formula is not exact for large s).
 * nint(sqrt(s)) = r+1 if s > r^2 + r else r, where r = floor(sqrt(s)):
 * sqrt(s) >= r + 1/2  <=>  s >= r^2 + r + 1/4  <=>  s > r^2 + r (integers).
 * ------------------------------------------------------------------------- */
int64_t oracle_isqrt(int64_t s)
{
    int64_t r = (int64_t)sqrt((double)s);
    while (r > 0 && r * r > s) r--;
    while ((r + 1) * (r + 1) <= s) r++;
    return r;
}

int64_t oracle_nint_sqrt(int64_t s)
{
    int64_t r = oracle_isqrt(s);
    return (s > r * r + r) ? r + 1 : r;
}

int64_t oracle_dist(int64_t xa, int64_t ya, int64_t xb, int64_t yb)
{
    int64_t dx = xa - xb, dy = ya - yb;
    return oracle_nint_sqrt(dx * dx + dy * dy);
}

/* d(tour[a], tour[b]) with positions taken modulo n: position n is position 0,
 * the closed tour of L18 Fig. 6 ("ordered coordinates") -- reading R10. */
static int64_t dpos(const int32_t *xy, const int32_t *tour, int64_t n,
                    int64_t a, int64_t b)
{
    int64_t ca = tour[a % n], cb = tour[b % n];
    return oracle_dist(xy[2 * ca], xy[2 * ca + 1], xy[2 * cb], xy[2 * cb + 1]);
}

/* Tour length: sum of the n closing edges d(t[k], t[k+1 mod n]). */
int64_t oracle_tour_length(const int32_t *xy, int64_t n, const int32_t *tour)
{
    int64_t L = 0;
    for (int64_t k = 0; k < n; k++) L += dpos(xy, tour, n, k, k + 1);
    return L;
}

/* 2-opt delta of pair (i, j), 0 <= i < j <= n-1 (north_star; L12 Fig. 2
 * "distance(b,f) + distance(g,d) > distance(b,d) + distance(g,f)" with
 * b = t[i], f = t[i+1], d = t[j], g = t[j+1]; reading R2):
 *   delta = d(i,j) + d(i+1,j+1) - d(i,i+1) - d(j,j+1);  improving iff < 0. */
int64_t oracle_delta(const int32_t *xy, int64_t n, const int32_t *tour,
                     int64_t i, int64_t j)
{
    return dpos(xy, tour, n, i, j) + dpos(xy, tour, n, i + 1, j + 1)
         - dpos(xy, tour, n, i, i + 1) - dpos(xy, tour, n, j, j + 1);
}

/* Fig. 3 cell number of pair (i, j), i < j: cells are numbered column by
 * column, "0,1 0  0,2 1  1,2 2  0,3 3 ..." (L14), i.e. k = j(j-1)/2 + i. */
int64_t oracle_cell(int64_t i, int64_t j) { return j * (j - 1) / 2 + i; }

/* ---------------------------------------------------------------------------
 * One exhaustive sweep (L14 Alg. 2 steps 2-5: "Calculate swap effect of one
 * pair ... Find the best value").  Neighbourhood: all pairs 0 <= i < j <= n-1
 * of the closed tour (reading R1, C(n,2) checks).  Best = lowest delta, ties
 * to the lowest Fig. 3 cell number (reading R5).  Scanning j ascending, then
 * i ascending, visits cells in increasing k, so a strict '<' keeps the lowest
 * cell among equal deltas.  At a 2-opt local minimum the winner is pair
 * (0, 1) with delta 0 (cell 0, a degenerate pair; reading R7).
 *
 * OpenMP splits the j loop; each thread keeps its own (delta, k) minimum and
 * the minima are combined with the same total order, which is independent of
 * the split.
 * ------------------------------------------------------------------------- */
void oracle_best_move(const int32_t *xy, int64_t n, const int32_t *tour,
                      int64_t *bi, int64_t *bj, int64_t *bdelta)
{
    int64_t best_d = 0, best_i = 0, best_j = 1;   /* pair (0,1): delta == 0 */
    /* route-ordered coordinates P[k] = coords[t[k]], P[n] = P[0] (L18 Fig. 6) */
    int64_t *px = (int64_t *)malloc(sizeof(int64_t) * (n + 1));
    int64_t *py = (int64_t *)malloc(sizeof(int64_t) * (n + 1));
    int64_t *e = (int64_t *)malloc(sizeof(int64_t) * n);
    for (int64_t k = 0; k <= n; k++) {
        int64_t c = tour[k % n];
        px[k] = xy[2 * c];
        py[k] = xy[2 * c + 1];
    }
    for (int64_t k = 0; k < n; k++) e[k] = oracle_dist(px[k], py[k], px[k + 1], py[k + 1]);

#pragma omp parallel
    {
        int64_t td = 0, ti = 0, tj = 1;
#pragma omp for schedule(dynamic, 16) nowait
        for (int64_t j = 1; j < n; j++) {
            for (int64_t i = 0; i < j; i++) {
                int64_t d = oracle_dist(px[i], py[i], px[j], py[j])
                          + oracle_dist(px[i + 1], py[i + 1], px[j + 1], py[j + 1])
                          - e[i] - e[j];
                if (d < td || (d == td && oracle_cell(i, j) < oracle_cell(ti, tj))) {
                    td = d; ti = i; tj = j;
                }
            }
        }
#pragma omp critical
        {
            if (td < best_d || (td == best_d && oracle_cell(ti, tj) < oracle_cell(best_i, best_j))) {
                best_d = td; best_i = ti; best_j = tj;
            }
        }
    }
    free(px); free(py); free(e);
    *bi = best_i; *bj = best_j; *bdelta = best_d;
}

/* The same argmin restricted to a list of rectangular tiles of the pair
 * matrix (L18 §IV.B problem division; L20 Fig. 7 "It is possible to calculate
 * distances in arbitrary segments"): tile t covers rows [I0, min(I0+TI, n-1)) x
 * columns [J0, min(J0+TJ, n)), pairs i < j only.  Used to check a shard of
 * the multi-GPU split.  Returns (0, 1, 0) if no pair in the tiles beats it. */
void oracle_best_move_tiles(const int32_t *xy, int64_t n, const int32_t *tour, const int32_t *tiles,
                            int64_t ntiles, int64_t TI, int64_t TJ, int64_t *bi, int64_t *bj, int64_t *bdelta)
{
    int64_t best_d = 0, best_i = 0, best_j = 1;
    for (int64_t t = 0; t < ntiles; t++) {
        int64_t I0 = tiles[2 * t], J0 = tiles[2 * t + 1];
        int64_t I1 = I0 + TI < n - 1 ? I0 + TI : n - 1, J1 = J0 + TJ < n ? J0 + TJ : n;
        for (int64_t j = J0; j < J1; j++)
            for (int64_t i = I0; i < I1 && i < j; i++) {
                int64_t d = oracle_delta(xy, n, tour, i, j);
                if (d < best_d || (d == best_d && oracle_cell(i, j) < oracle_cell(best_i, best_j))) {
                    best_d = d; best_i = i; best_j = j;
                }
            }
    }
    *bi = best_i; *bj = best_j; *bdelta = best_d;
}

/* The 2-opt move (L12 §I.B "removes two edges ... reconnects ... reversing
 * order of sub-tour"; Fig. 1): reverse tour positions i+1..j (reading R6:
 * never the complement, so tour[0] never moves). */
void oracle_apply(int32_t *tour, int64_t i, int64_t j)
{
    for (int64_t a = i + 1, b = j; a < b; a++, b--) {
        int32_t t = tour[a]; tour[a] = tour[b]; tour[b] = t;
    }
}

/* Best-improvement 2-opt local search (L12: "This step is applied only if the
 * new tour would be shorter. Repeating removing and reconnecting the tour until
 * no 2-opt improvements can be found leads to ... (local minimum)").
 * Returns 0 at a local minimum, 1 when max_iters moves were applied first
 * (max_iters < 0: unbounded).  trace (may be NULL) receives (i, j, delta) of
 * every applied move, up to trace_cap moves. */
int oracle_local_search(const int32_t *xy, int64_t n, int32_t *tour, int64_t max_iters,
                        int64_t *length, int64_t *iterations,
                        int64_t *trace, int64_t trace_cap)
{
    int64_t L = oracle_tour_length(xy, n, tour);
    int64_t it = 0;
    int status = 0;
    for (;;) {
        if (max_iters >= 0 && it >= max_iters) {
            /* reading R8: report MAXITER only if an improving move remains */
            int64_t i, j, d;
            oracle_best_move(xy, n, tour, &i, &j, &d);
            status = (d < 0) ? 1 : 0;
            break;
        }
        int64_t i, j, d;
        oracle_best_move(xy, n, tour, &i, &j, &d);
        if (d >= 0) break;
        oracle_apply(tour, i, j);
        L += d;
        if (trace && it < trace_cap) {
            trace[3 * it] = i; trace[3 * it + 1] = j; trace[3 * it + 2] = d;
        }
        it++;
    }
    *length = L;
    *iterations = it;
    return status;
}

/* ---------------------------------------------------------------------------
 * Iterated Local Search (L10 Algorithm 1: s0 = GenerateInitialSolution();
 * s* = 2optLocalSearch(s0); while not terminated: s' = Perturbation(s*);
 * s*' = 2optLocalSearch(s'); s* = AcceptanceCriterion(s*, s*')), with the
 * paper's choices (L18 §V): a random initial tour (the caller's), "a simple
 * doublebridge move as a perturbation technique".  Readings (DESIGN.md §3,
 * R14-R16): termination = a fixed number of iterations; acceptance = keep the
 * new local minimum iff it is strictly shorter; the double bridge of the
 * current tour t = A B C D (cut positions 1 <= a < b < c <= n-1, tour[0] in A)
 * is A C B D, with segment lengths drawn from the counter-based splitmix64
 * stream of `seed` (draw k of iteration it is output 3*it + k):
 *   len_k = 1 + out % max(1, (n - 1) / 3),  a = len_0, b = a + len_1, c = b + len_2.
 * ------------------------------------------------------------------------- */
static uint64_t oracle_splitmix64_at(uint64_t seed, uint64_t k)
{
    /* output k (0-based) of splitmix64 seeded with `seed` (Steele, Lea, Flood) */
    uint64_t z = seed + (k + 1) * 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

void oracle_double_bridge_cuts(int64_t n, uint64_t seed, int64_t it, int64_t *a, int64_t *b, int64_t *c)
{
    int64_t m = (n - 1) / 3;
    if (m < 1) m = 1;
    int64_t l0 = 1 + (int64_t)(oracle_splitmix64_at(seed, 3 * (uint64_t)it) % (uint64_t)m);
    int64_t l1 = 1 + (int64_t)(oracle_splitmix64_at(seed, 3 * (uint64_t)it + 1) % (uint64_t)m);
    int64_t l2 = 1 + (int64_t)(oracle_splitmix64_at(seed, 3 * (uint64_t)it + 2) % (uint64_t)m);
    *a = l0;
    *b = l0 + l1;
    *c = l0 + l1 + l2;
}

/* out = A C B D for tour = A B C D with A = [0, a), B = [a, b), C = [b, c), D = [c, n) */
void oracle_double_bridge(const int32_t *tour, int64_t n, int64_t a, int64_t b, int64_t c, int32_t *out)
{
    int64_t k = 0;
    for (int64_t p = 0; p < a; p++) out[k++] = tour[p];
    for (int64_t p = b; p < c; p++) out[k++] = tour[p];
    for (int64_t p = a; p < b; p++) out[k++] = tour[p];
    for (int64_t p = c; p < n; p++) out[k++] = tour[p];
}

/* Runs `iterations` ILS steps from `tour` (in: start tour; out: best tour).
 * lengths (may be NULL) receives the current best length after each step
 * (lengths[0] = the first local minimum, lengths[t+1] after step t). */
void oracle_ils(const int32_t *xy, int64_t n, int32_t *tour, int64_t iterations, uint64_t seed,
                int64_t *length, int64_t *lengths)
{
    int64_t L, it;
    oracle_local_search(xy, n, tour, -1, &L, &it, NULL, 0);
    if (lengths) lengths[0] = L;
    int32_t *cand = (int32_t *)malloc(sizeof(int32_t) * n);
    for (int64_t t = 0; t < iterations; t++) {
        if (n >= 8) {
            int64_t a, b, c, L2, it2;
            oracle_double_bridge_cuts(n, seed, t, &a, &b, &c);
            oracle_double_bridge(tour, n, a, b, c, cand);
            oracle_local_search(xy, n, cand, -1, &L2, &it2, NULL, 0);
            if (L2 < L) {
                memcpy(tour, cand, sizeof(int32_t) * n);
                L = L2;
            }
        }
        if (lengths) lengths[t + 1] = L;
    }
    free(cand);
    *length = L;
}

/* ---------------------------------------------------------------------------
 * Multiple Fragment (greedy) start tour.  L22 §V: "an initial solution based
 * on the Multiple Fragment(Greedy) heuristic[18]"; the paper gives no more
 * than the name, so reading R17 fixes the textbook definition:
 * take the edges {u, v} in increasing order of (d(u,v), min(u,v), max(u,v))
 * and keep an edge iff both ends have degree < 2 and it does not close a
 * cycle; the n-1 kept edges form a Hamiltonian path, closed by the edge
 * between its two ends.  Tour: start at city 0, step to its lower-id
 * neighbour, then follow the cycle.  Plain version: all C(n,2) edges, one
 * sort, union-find -- O(n^2 log n) time and 8 C(n,2) bytes (4.6 GB at n = 33810,
 * 29.5 GB at n = 85900; golden files only).  Returns 0, or -1 if n is out of
 * range [3, 2^22] or memory runs out.
 * ------------------------------------------------------------------------- */
static int cmp_u64(const void *a, const void *b)
{
    uint64_t x = *(const uint64_t *)a, y = *(const uint64_t *)b;
    return x < y ? -1 : x > y;
}

static int64_t uf_find(int64_t *parent, int64_t x)
{
    while (parent[x] != x) {
        parent[x] = parent[parent[x]];
        x = parent[x];
    }
    return x;
}

int oracle_mf_tour(const int32_t *xy, int64_t n, int32_t *tour)
{
    if (n < 3 || n > (1 << 22)) return -1; /* key packing below; memory: 4 n(n-1) bytes */
    const int64_t m = n * (n - 1) / 2;
    uint64_t *key = (uint64_t *)malloc(sizeof(uint64_t) * m);
    int64_t *parent = (int64_t *)malloc(sizeof(int64_t) * n);
    int64_t *adj = (int64_t *)malloc(sizeof(int64_t) * 2 * n);
    int32_t *deg = (int32_t *)calloc(n, sizeof(int32_t));
    if (!key || !parent || !adj || !deg) {
        free(key), free(parent), free(adj), free(deg);
        return -1;
    }
    int64_t e = 0;
    for (int64_t v = 1; v < n; v++)
        for (int64_t u = 0; u < v; u++) {
            const uint64_t d = (uint64_t)oracle_dist(xy[2 * u], xy[2 * u + 1], xy[2 * v], xy[2 * v + 1]);
            key[e++] = d << 44 | (uint64_t)u << 22 | (uint64_t)v;  /* d < 2^17, u < v < 2^22 */
        }
    qsort(key, m, sizeof(uint64_t), cmp_u64);
    for (int64_t k = 0; k < n; k++) parent[k] = k;
    int64_t kept = 0;
    for (int64_t t = 0; t < m && kept < n - 1; t++) {
        const int64_t u = (int64_t)(key[t] >> 22 & 0x3FFFFF), v = (int64_t)(key[t] & 0x3FFFFF);
        if (deg[u] >= 2 || deg[v] >= 2) continue;
        const int64_t ru = uf_find(parent, u), rv = uf_find(parent, v);
        if (ru == rv) continue; /* would close a cycle */
        parent[ru] = rv;
        adj[2 * u + deg[u]++] = v;
        adj[2 * v + deg[v]++] = u;
        kept++;
    }
    /* close the Hamiltonian path: its two ends are the cities of degree 1 */
    int64_t a = -1, b = -1;
    for (int64_t k = 0; k < n; k++)
        if (deg[k] < 2) {
            if (a < 0) a = k;
            else b = k;
        }
    adj[2 * a + deg[a]++] = b;
    adj[2 * b + deg[b]++] = a;
    /* walk: 0, then its lower-id neighbour */
    int64_t prev = 0, cur = adj[0] < adj[1] ? adj[0] : adj[1];
    tour[0] = 0;
    for (int64_t k = 1; k < n; k++) {
        tour[k] = (int32_t)cur;
        const int64_t next = adj[2 * cur] == prev ? adj[2 * cur + 1] : adj[2 * cur];
        prev = cur;
        cur = next;
    }
    free(key), free(parent), free(adj), free(deg);
    return 0;
}

int oracle_num_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* ---------------------------------------------------------------------------
 * Neighbourhood-pruned best-improvement 2-opt.
 * L18 §V: "Possibly limiting the neighborhood would also bring an improvement
 * in efficiency"; L26 §VII: "simple ideas such as neighborhood pruning can be
 * applied at the cost of the quality of the solution".  The paper names the
 * idea only; reading R18 fixes the textbook K-nearest-neighbour
 * candidate rule:
 *   N_K(a)  = the K cities c != a with the smallest (d(a,c), c);
 *   E_K     = { {a,c} : c in N_K(a) or a in N_K(c) };
 *   M_K     = the 2-opt pairs (i, j), 0 <= i < j <= n-1 of the closed tour,
 *             with {t[i], t[j]} in E_K or {t[i+1], t[j+1]} in E_K
 *             (a move is kept iff one of the two edges it creates joins
 *             candidate neighbours).
 * The best move is the lowest (delta, Fig. 3 cell) over the pairs of M_K with
 * delta < 0, else (0, 1, 0) (reading R7).  K >= n-1 gives the full
 * neighbourhood (every pair), i.e. oracle_best_move.
 * ------------------------------------------------------------------------- */

/* N_K by plain selection: for every city, keep the K smallest (d, id) of all
 * other cities by insertion into a sorted list.  nbr[a*K + r] = r-th nearest,
 * -1 where n-1 < K. */
void oracle_knn(const int32_t *xy, int64_t n, int64_t K, int32_t *nbr)
{
#pragma omp parallel for schedule(dynamic, 64)
    for (int64_t a = 0; a < n; a++) {
        int64_t *bd = (int64_t *)malloc(sizeof(int64_t) * K);
        int32_t *bc = (int32_t *)malloc(sizeof(int32_t) * K);
        int64_t cnt = 0;
        for (int64_t c = 0; c < n; c++) {
            if (c == a) continue;
            int64_t d = oracle_dist(xy[2 * a], xy[2 * a + 1], xy[2 * c], xy[2 * c + 1]);
            if (cnt == K && d >= bd[K - 1]) continue; /* ids ascend: (d, c) > the K-th */
            int64_t r = cnt < K ? cnt++ : K - 1;
            while (r > 0 && bd[r - 1] > d) { /* equal d: the earlier (lower) id stays first */
                bd[r] = bd[r - 1];
                bc[r] = bc[r - 1];
                r--;
            }
            bd[r] = d;
            bc[r] = (int32_t)c;
        }
        for (int64_t r = 0; r < K; r++) nbr[a * K + r] = r < cnt ? bc[r] : -1;
        free(bd);
        free(bc);
    }
}

/* {a, c} in E_K */
static int in_candidate_edges(const int32_t *nbr, int64_t K, int64_t a, int64_t c)
{
    for (int64_t r = 0; r < K; r++)
        if (nbr[a * K + r] == c || nbr[c * K + r] == a) return 1;
    return 0;
}

/* Plain form: every pair of the full sweep in Fig. 3 order, kept iff in M_K. */
void oracle_pruned_best_move_plain(const int32_t *xy, int64_t n, const int32_t *tour, const int32_t *nbr,
                                   int64_t K, int64_t *bi, int64_t *bj, int64_t *bdelta)
{
    int64_t best_d = 0, best_i = 0, best_j = 1;
#pragma omp parallel
    {
        int64_t td = 0, ti = 0, tj = 1;
#pragma omp for schedule(dynamic, 16) nowait
        for (int64_t j = 1; j < n; j++) {
            for (int64_t i = 0; i < j; i++) {
                if (!in_candidate_edges(nbr, K, tour[i], tour[j]) &&
                    !in_candidate_edges(nbr, K, tour[i + 1], tour[(j + 1) % n]))
                    continue;
                int64_t d = oracle_delta(xy, n, tour, i, j);
                if (d < td || (d == td && oracle_cell(i, j) < oracle_cell(ti, tj))) {
                    td = d; ti = i; tj = j;
                }
            }
        }
#pragma omp critical
        {
            if (td < best_d || (td == best_d && oracle_cell(ti, tj) < oracle_cell(best_i, best_j))) {
                best_d = td; best_i = ti; best_j = tj;
            }
        }
    }
    *bi = best_i; *bj = best_j; *bdelta = best_d;
}

/* The same set M_K enumerated from the candidate lists, O(nK) per sweep: for
 * every candidate edge {a, c} (a at position p, c at position q, u < v the two
 * positions), the two moves that create it are
 *   (u, v)        -- {t[i], t[j]} = {a, c}, and
 *   (u-1, v-1)    -- {t[i+1], t[j+1]} = {a, c}; for u = 0 position 0 is
 *                    position n of the closed tour, giving (v-1, n-1).
 * Pinned to oracle_pruned_best_move_plain (tests/test_oracle_pruned.py). */
void oracle_pruned_best_move(const int32_t *xy, int64_t n, const int32_t *tour, const int32_t *nbr, int64_t K,
                             int64_t *bi, int64_t *bj, int64_t *bdelta)
{
    int64_t best_d = 0, best_i = 0, best_j = 1;
    int64_t *pos = (int64_t *)malloc(sizeof(int64_t) * n);
    for (int64_t k = 0; k < n; k++) pos[tour[k]] = k;
#pragma omp parallel
    {
        int64_t td = 0, ti = 0, tj = 1;
#pragma omp for schedule(static) nowait
        for (int64_t p = 0; p < n; p++) {
            const int64_t a = tour[p];
            for (int64_t r = 0; r < K; r++) {
                const int64_t c = nbr[a * K + r];
                if (c < 0) continue;
                const int64_t q = pos[c];
                const int64_t u = p < q ? p : q, v = p < q ? q : p;
                const int64_t cand[2][2] = {{u, v}, {u >= 1 ? u - 1 : v - 1, u >= 1 ? v - 1 : n - 1}};
                for (int m = 0; m < 2; m++) {
                    const int64_t i = cand[m][0], j = cand[m][1];
                    const int64_t d = oracle_delta(xy, n, tour, i, j);
                    if (d < td || (d == td && oracle_cell(i, j) < oracle_cell(ti, tj))) {
                        td = d; ti = i; tj = j;
                    }
                }
            }
        }
#pragma omp critical
        {
            if (td < best_d || (td == best_d && oracle_cell(ti, tj) < oracle_cell(best_i, best_j))) {
                best_d = td; best_i = ti; best_j = tj;
            }
        }
    }
    free(pos);
    *bi = best_i; *bj = best_j; *bdelta = best_d;
}

/* First improvement over M_K (readings R18 + R20): the pair of M_K with
 * delta < 0 and the lowest Fig. 3 cell, scanning the pairs in cell order. */
void oracle_pruned_first_move(const int32_t *xy, int64_t n, const int32_t *tour, const int32_t *nbr, int64_t K,
                              int64_t *bi, int64_t *bj, int64_t *bdelta)
{
    for (int64_t j = 1; j < n; j++)
        for (int64_t i = 0; i < j; i++) {
            if (!in_candidate_edges(nbr, K, tour[i], tour[j]) &&
                !in_candidate_edges(nbr, K, tour[i + 1], tour[(j + 1) % n]))
                continue;
            int64_t d = oracle_delta(xy, n, tour, i, j);
            if (d < 0) {
                *bi = i; *bj = j; *bdelta = d;
                return;
            }
        }
    *bi = 0; *bj = 1; *bdelta = 0;
}

/* Local search over M_K (same loop, status and trace conventions as
 * oracle_local_search).  mode bit 0: the plain all-pairs scan instead of the
 * list enumeration (best improvement); bit 1: first improvement (R20). */
int oracle_pruned_local_search(const int32_t *xy, int64_t n, int32_t *tour, int64_t K, int64_t max_iters, int mode,
                               int64_t *length, int64_t *iterations, int64_t *trace, int64_t trace_cap)
{
    int32_t *nbr = (int32_t *)malloc(sizeof(int32_t) * n * K);
    oracle_knn(xy, n, K, nbr);
    int64_t L = oracle_tour_length(xy, n, tour);
    int64_t it = 0;
    int status = 0;
    for (;;) {
        int64_t i, j, d;
        if (mode & 2) oracle_pruned_first_move(xy, n, tour, nbr, K, &i, &j, &d);
        else if (mode & 1) oracle_pruned_best_move_plain(xy, n, tour, nbr, K, &i, &j, &d);
        else oracle_pruned_best_move(xy, n, tour, nbr, K, &i, &j, &d);
        if (d >= 0) break;
        if (max_iters >= 0 && it >= max_iters) { /* reading R8 */
            status = 1;
            break;
        }
        oracle_apply(tour, i, j);
        L += d;
        if (trace && it < trace_cap) {
            trace[3 * it] = i; trace[3 * it + 1] = j; trace[3 * it + 2] = d;
        }
        it++;
    }
    free(nbr);
    *length = L;
    *iterations = it;
    return status;
}

/* ---------------------------------------------------------------------------
 * 2.5-opt (2h-opt): best-improvement 2-opt plus node insertion (SURVEY.md
 * §8(f) NEXT-4).  L26 §VII: "Our future work is to efficiently implement more
 * complex local search algorithms such as 2.5-opt"; the paper gives no
 * definition, so reading R19 takes the textbook 2h-opt
 * neighbourhood over the same pairs 0 <= i < j <= n-1 of the closed tour as
 * the 2-opt sweep (reading R1), three moves per pair:
 *   type 0  the 2-opt move (reverse positions i+1..j);
 *   type 1  (j >= i+2) move city t[i+1] between t[j] and t[j+1]:
 *           delta = d(t_i, t_{i+2}) - e_i - e_{i+1} + d(t_j, t_{i+1}) + d(t_{i+1}, t_{j+1}) - e_j;
 *   type 2  (j >= i+2) move city t[j] between t[i] and t[i+1]:
 *           delta = d(t_{j-1}, t_{j+1}) - e_{j-1} - e_j + d(t_i, t_j) + d(t_j, t_{i+1}) - e_i.
 * Best = the lowest (delta, Fig. 3 cell, type) with delta < 0, else
 * (0, 1, type 0, delta 0).  Positions i+1..j are the only ones that move:
 * type 1 rotates them left by one, type 2 right by one, so t[0] never moves
 * (reading R6) and every city but t[0] can be inserted into every edge that
 * does not touch it.
 * ------------------------------------------------------------------------- */
int64_t oracle25_delta(const int32_t *xy, int64_t n, const int32_t *tour, int64_t i, int64_t j, int type)
{
    if (type == 0) return oracle_delta(xy, n, tour, i, j);
    if (j < i + 2) return INT64_MAX; /* not a move */
    if (type == 1)
        return dpos(xy, tour, n, i, i + 2) - dpos(xy, tour, n, i, i + 1) - dpos(xy, tour, n, i + 1, i + 2)
             + dpos(xy, tour, n, j, i + 1) + dpos(xy, tour, n, i + 1, j + 1) - dpos(xy, tour, n, j, j + 1);
    return dpos(xy, tour, n, j - 1, j + 1) - dpos(xy, tour, n, j - 1, j) - dpos(xy, tour, n, j, j + 1)
         + dpos(xy, tour, n, i, j) + dpos(xy, tour, n, j, i + 1) - dpos(xy, tour, n, i, i + 1);
}

/* One exhaustive 2.5-opt sweep.  Same terms as oracle25_delta, computed once
 * per sweep: route-ordered coordinates, edges e_k and removal gains
 * g_k = d(t_{k-1}, t_{k+1}) - e_{k-1} - e_k; per pair the three distances
 * d(i,j), d(i+1,j+1), d(i+1,j).  Pinned to oracle25_delta and to a brute
 * force over explicitly built neighbours (tests/test_oracle_25opt.py). */
void oracle25_best_move(const int32_t *xy, int64_t n, const int32_t *tour,
                        int64_t *bi, int64_t *bj, int64_t *btype, int64_t *bdelta)
{
    int64_t best_d = 0, best_i = 0, best_j = 1, best_t = 0;
    int64_t *px = (int64_t *)malloc(sizeof(int64_t) * (n + 1));
    int64_t *py = (int64_t *)malloc(sizeof(int64_t) * (n + 1));
    int64_t *e = (int64_t *)malloc(sizeof(int64_t) * n);
    int64_t *g = (int64_t *)malloc(sizeof(int64_t) * n);
    for (int64_t k = 0; k <= n; k++) {
        int64_t c = tour[k % n];
        px[k] = xy[2 * c];
        py[k] = xy[2 * c + 1];
    }
    for (int64_t k = 0; k < n; k++) e[k] = oracle_dist(px[k], py[k], px[k + 1], py[k + 1]);
    for (int64_t k = 0; k < n; k++) {
        int64_t km = (k + n - 1) % n;
        g[k] = oracle_dist(px[km], py[km], px[k + 1], py[k + 1]) - e[km] - e[k];
    }
#pragma omp parallel
    {
        int64_t td = 0, ti = 0, tj = 1, tt = 0;
#pragma omp for schedule(dynamic, 16) nowait
        for (int64_t j = 1; j < n; j++) {
            for (int64_t i = 0; i < j; i++) {
                const int64_t dij = oracle_dist(px[i], py[i], px[j], py[j]);
                const int64_t di1j1 = oracle_dist(px[i + 1], py[i + 1], px[j + 1], py[j + 1]);
                int64_t d[3] = {dij + di1j1 - e[i] - e[j], INT64_MAX, INT64_MAX};
                if (j >= i + 2) {
                    const int64_t di1j = oracle_dist(px[i + 1], py[i + 1], px[j], py[j]);
                    d[1] = g[i + 1] + di1j + di1j1 - e[j];
                    d[2] = g[j] + dij + di1j - e[i];
                }
                for (int t = 0; t < 3; t++) {
                    /* visiting (cell, type) in increasing order: strict '<' keeps the lowest */
                    if (d[t] < td || (d[t] == td && (oracle_cell(i, j) < oracle_cell(ti, tj) ||
                                                     (oracle_cell(i, j) == oracle_cell(ti, tj) && t < tt)))) {
                        td = d[t]; ti = i; tj = j; tt = t;
                    }
                }
            }
        }
#pragma omp critical
        {
            if (td < best_d || (td == best_d && (oracle_cell(ti, tj) < oracle_cell(best_i, best_j) ||
                                                 (oracle_cell(ti, tj) == oracle_cell(best_i, best_j) && tt < best_t)))) {
                best_d = td; best_i = ti; best_j = tj; best_t = tt;
            }
        }
    }
    free(px); free(py); free(e); free(g);
    *bi = best_i; *bj = best_j; *btype = best_t; *bdelta = best_d;
}

/* Apply move (i, j, type): type 0 reverses positions i+1..j; type 1 moves
 * t[i+1] to position j (positions i+2..j shift left); type 2 moves t[j] to
 * position i+1 (positions i+1..j-1 shift right). */
void oracle25_apply(int32_t *tour, int64_t i, int64_t j, int type)
{
    if (type == 0) {
        oracle_apply(tour, i, j);
    } else if (type == 1) {
        int32_t c = tour[i + 1];
        for (int64_t k = i + 1; k < j; k++) tour[k] = tour[k + 1];
        tour[j] = c;
    } else {
        int32_t c = tour[j];
        for (int64_t k = j; k > i + 1; k--) tour[k] = tour[k - 1];
        tour[i + 1] = c;
    }
}

/* Best-improvement 2.5-opt local search; trace rows (i, j, delta, type). */
int oracle25_local_search(const int32_t *xy, int64_t n, int32_t *tour, int64_t max_iters,
                          int64_t *length, int64_t *iterations, int64_t *trace, int64_t trace_cap)
{
    int64_t L = oracle_tour_length(xy, n, tour);
    int64_t it = 0;
    int status = 0;
    for (;;) {
        int64_t i, j, t, d;
        oracle25_best_move(xy, n, tour, &i, &j, &t, &d);
        if (d >= 0) break;
        if (max_iters >= 0 && it >= max_iters) { /* reading R8 */
            status = 1;
            break;
        }
        oracle25_apply(tour, i, j, (int)t);
        L += d;
        if (trace && it < trace_cap) {
            trace[4 * it] = i; trace[4 * it + 1] = j; trace[4 * it + 2] = d; trace[4 * it + 3] = t;
        }
        it++;
    }
    *length = L;
    *iterations = it;
    return status;
}

/* ---------------------------------------------------------------------------
 * First-improvement 2-opt.  Reading R20 (DESIGN.md
 * §3): the paper's sequential loop visits the pairs in the Fig. 3 cell order
 * (L14: "0,1 0  0,2 1  1,2 2 ..."); first improvement applies the first pair
 * of that order with delta < 0 and restarts the scan, i.e. it takes the
 * improving pair with the lowest cell number instead of the lowest delta.
 * Same neighbourhood (reading R1), same apply, same termination (R7): at a
 * local minimum it returns (0, 1, 0).
 * ------------------------------------------------------------------------- */
void oracle_first_move(const int32_t *xy, int64_t n, const int32_t *tour, int64_t *bi, int64_t *bj, int64_t *bdelta)
{
    for (int64_t j = 1; j < n; j++)
        for (int64_t i = 0; i < j; i++) {
            int64_t d = oracle_delta(xy, n, tour, i, j);
            if (d < 0) {
                *bi = i; *bj = j; *bdelta = d;
                return;
            }
        }
    *bi = 0; *bj = 1; *bdelta = 0;
}

int oracle_first_local_search(const int32_t *xy, int64_t n, int32_t *tour, int64_t max_iters,
                              int64_t *length, int64_t *iterations, int64_t *trace, int64_t trace_cap)
{
    int64_t L = oracle_tour_length(xy, n, tour);
    int64_t it = 0;
    int status = 0;
    for (;;) {
        int64_t i, j, d;
        oracle_first_move(xy, n, tour, &i, &j, &d);
        if (d >= 0) break;
        if (max_iters >= 0 && it >= max_iters) { /* reading R8 */
            status = 1;
            break;
        }
        oracle_apply(tour, i, j);
        L += d;
        if (trace && it < trace_cap) {
            trace[3 * it] = i; trace[3 * it + 1] = j; trace[3 * it + 2] = d;
        }
        it++;
    }
    *length = L;
    *iterations = it;
    return status;
}


/* ---------------------------------------------------------------------------
 * Iterated Local Search over any of the local searches above (L10 Algorithm 1
 * with "2optLocalSearch" replaced by the variant; L26 §VII names 2.5-opt as
 * the next local search).  Same perturbation, acceptance and termination as
 * oracle_ils (readings R14-R16).  mode: 0 best-improvement 2-opt (== oracle_ils),
 * 1 pruned to K neighbours (R18), 2 first improvement (R20), 3 pruned + first,
 * 4 2.5-opt (R19).
 * ------------------------------------------------------------------------- */
static void ls_mode(const int32_t *xy, int64_t n, int32_t *tour, int mode, int64_t K, int64_t *L)
{
    int64_t it;
    if (mode == 0) oracle_local_search(xy, n, tour, -1, L, &it, NULL, 0);
    else if (mode == 1) oracle_pruned_local_search(xy, n, tour, K, -1, 0, L, &it, NULL, 0);
    else if (mode == 2) oracle_first_local_search(xy, n, tour, -1, L, &it, NULL, 0);
    else if (mode == 3) oracle_pruned_local_search(xy, n, tour, K, -1, 2, L, &it, NULL, 0);
    else oracle25_local_search(xy, n, tour, -1, L, &it, NULL, 0);
}

void oracle_ils_mode(const int32_t *xy, int64_t n, int32_t *tour, int64_t iterations, uint64_t seed, int mode,
                     int64_t K, int64_t *length, int64_t *lengths)
{
    int64_t L;
    ls_mode(xy, n, tour, mode, K, &L);
    if (lengths) lengths[0] = L;
    int32_t *cand = (int32_t *)malloc(sizeof(int32_t) * n);
    for (int64_t t = 0; t < iterations; t++) {
        if (n >= 8) {
            int64_t a, b, c, L2;
            oracle_double_bridge_cuts(n, seed, t, &a, &b, &c);
            oracle_double_bridge(tour, n, a, b, c, cand);
            ls_mode(xy, n, cand, mode, K, &L2);
            if (L2 < L) {
                memcpy(tour, cand, sizeof(int32_t) * n);
                L = L2;
            }
        }
        if (lengths) lengths[t + 1] = L;
    }
    free(cand);
    *length = L;
}

/* ---------------------------------------------------------------------------
 * Or-opt ("2.5-opt/Or-opt variants"; L18 §V "more
 * sophisticated algorithms such as 3-opt, k-opt or LK"; L26 §VII "2.5-opt,
 * 3-opt and Lin-Kernighan").  The paper gives no definition; reading R21
 * takes Or's textbook neighbourhood -- 2-opt plus moving a
 * segment of L = 1, 2 or 3 consecutive cities, in either orientation, into
 * another edge -- over the same pairs 0 <= i < j <= n-1 as the 2-opt sweep
 * (reading R1).  Types (13 per pair):
 *   type 0                     the 2-opt move (reverse positions i+1..j);
 *   type 1 + 4(L-1) + 2 dir + rev, for j >= i+L+1:
 *     dir 0 (forward):  segment t[i+1..i+L] moves between t[j] and t[j+1];
 *     dir 1 (backward): segment t[j-L+1..j] moves between t[i] and t[i+1];
 *     rev 1: the segment is inserted reversed.
 * With a = the segment's first city and b its last (rev swaps them):
 *   forward:  delta = d(t_i, t_{i+L+1}) - d(t_i, t_{i+1}) - d(t_{i+L}, t_{i+L+1})
 *                   + d(t_j, a) + d(b, t_{j+1}) - d(t_j, t_{j+1});
 *   backward: delta = d(t_{j-L}, t_{j+1}) - d(t_{j-L}, t_{j-L+1}) - d(t_j, t_{j+1})
 *                   + d(t_i, a) + d(b, t_{i+1}) - d(t_i, t_{i+1}).
 * L = 1 forward / backward are 2.5-opt's types 1 / 2 (reading R19); for
 * L = 1 the reversed types equal the plain ones and lose the type tie-break.
 * Best = the lowest (delta, Fig. 3 cell, type) with delta < 0, else
 * (0, 1, type 0, delta 0).  Only positions i+1..j move, so t[0] never moves
 * (reading R6): segments containing t[0] are not moved.
 * ------------------------------------------------------------------------- */
int64_t oracleor_delta(const int32_t *xy, int64_t n, const int32_t *tour, int64_t i, int64_t j, int type)
{
    if (type == 0) return oracle_delta(xy, n, tour, i, j);
    if (type < 0 || type > 12) return INT64_MAX;
    const int64_t L = 1 + (type - 1) / 4, dir = ((type - 1) / 2) & 1, rev = (type - 1) & 1;
    if (j < i + L + 1) return INT64_MAX; /* not a move */
    if (dir == 0) {
        const int64_t a = rev ? i + L : i + 1, b = rev ? i + 1 : i + L;
        return dpos(xy, tour, n, i, i + L + 1) - dpos(xy, tour, n, i, i + 1) - dpos(xy, tour, n, i + L, i + L + 1)
             + dpos(xy, tour, n, j, a) + dpos(xy, tour, n, b, j + 1) - dpos(xy, tour, n, j, j + 1);
    }
    const int64_t a = rev ? j : j - L + 1, b = rev ? j - L + 1 : j;
    return dpos(xy, tour, n, j - L, j + 1) - dpos(xy, tour, n, j - L, j - L + 1) - dpos(xy, tour, n, j, j + 1)
         + dpos(xy, tour, n, i, a) + dpos(xy, tour, n, b, i + 1) - dpos(xy, tour, n, i, i + 1);
}

/* One exhaustive Or-opt sweep: every (j, i, type) in increasing (cell, type)
 * order, oracleor_delta per move, strict '<' keeps the lowest. */
void oracleor_best_move(const int32_t *xy, int64_t n, const int32_t *tour,
                        int64_t *bi, int64_t *bj, int64_t *btype, int64_t *bdelta)
{
    int64_t best_d = 0, best_i = 0, best_j = 1, best_t = 0;
#pragma omp parallel
    {
        int64_t td = 0, ti = 0, tj = 1, tt = 0;
#pragma omp for schedule(dynamic, 16) nowait
        for (int64_t j = 1; j < n; j++)
            for (int64_t i = 0; i < j; i++)
                for (int t = 0; t <= 12; t++) {
                    const int64_t d = oracleor_delta(xy, n, tour, i, j, t);
                    if (d < td || (d == td && (oracle_cell(i, j) < oracle_cell(ti, tj) ||
                                               (oracle_cell(i, j) == oracle_cell(ti, tj) && t < tt)))) {
                        td = d; ti = i; tj = j; tt = t;
                    }
                }
#pragma omp critical
        {
            if (td < best_d || (td == best_d && (oracle_cell(ti, tj) < oracle_cell(best_i, best_j) ||
                                                 (oracle_cell(ti, tj) == oracle_cell(best_i, best_j) && tt < best_t)))) {
                best_d = td; best_i = ti; best_j = tj; best_t = tt;
            }
        }
    }
    *bi = best_i; *bj = best_j; *btype = best_t; *bdelta = best_d;
}

/* Apply move (i, j, type) by writing positions i+1..j in their new order:
 * the rest of the span first (forward) or last (backward), the segment in
 * its (possibly reversed) order in the edge it moves into. */
void oracleor_apply(int32_t *tour, int64_t i, int64_t j, int type)
{
    if (type == 0) {
        oracle_apply(tour, i, j);
        return;
    }
    const int64_t L = 1 + (type - 1) / 4, dir = ((type - 1) / 2) & 1, rev = (type - 1) & 1;
    const int64_t m = j - i;
    int32_t *span = (int32_t *)malloc(sizeof(int32_t) * m);
    int64_t w = 0;
    if (dir == 0) {
        for (int64_t k = i + L + 1; k <= j; k++) span[w++] = tour[k];
        for (int64_t q = 0; q < L; q++) span[w++] = tour[rev ? i + L - q : i + 1 + q];
    } else {
        for (int64_t q = 0; q < L; q++) span[w++] = tour[rev ? j - q : j - L + 1 + q];
        for (int64_t k = i + 1; k <= j - L; k++) span[w++] = tour[k];
    }
    memcpy(tour + i + 1, span, sizeof(int32_t) * m);
    free(span);
}

/* Best-improvement Or-opt local search; trace rows (i, j, delta, type). */
int oracleor_local_search(const int32_t *xy, int64_t n, int32_t *tour, int64_t max_iters,
                          int64_t *length, int64_t *iterations, int64_t *trace, int64_t trace_cap)
{
    int64_t L = oracle_tour_length(xy, n, tour);
    int64_t it = 0;
    int status = 0;
    for (;;) {
        int64_t i, j, t, d;
        oracleor_best_move(xy, n, tour, &i, &j, &t, &d);
        if (d >= 0) break;
        if (max_iters >= 0 && it >= max_iters) { /* reading R8 */
            status = 1;
            break;
        }
        oracleor_apply(tour, i, j, (int)t);
        L += d;
        if (trace && it < trace_cap) {
            trace[4 * it] = i; trace[4 * it + 1] = j; trace[4 * it + 2] = d; trace[4 * it + 3] = t;
        }
        it++;
    }
    *length = L;
    *iterations = it;
    return status;
}

/* ---------------------------------------------------------------------------
 * Exact radius-pruned sweeps (SURVEY.md §8(c) "Exact pruned oracle for large
 * n").  These return EXACTLY what the plain all-pairs sweeps above return --
 * they are not a different neighbourhood -- but visit only the pairs that can
 * improve, so whole C4/C5 local searches from a constructive start finish in
 * minutes instead of hours.  They exist to write golden traces at those sizes
 * (tests/golden/make_golden.py) and are pinned move by move against the plain
 * sweeps (tests/test_oracle_radius.py).
 *
 * Lemma (2-opt, L12 Fig. 2 delta, reading R2):
 *   delta(i,j) = [D(t_i,t_j) - e_i] + [D(t_{i+1},t_{j+1}) - e_j] < 0
 *   implies D(t_i,t_j) < e_i  or  D(t_{i+1},t_{j+1}) < e_j
 * (if both brackets are >= 0 the sum is >= 0).  So the improving pairs are
 * among
 *   (A) i = p, j = q > p       with D(t_p, t_q) < e_p, and
 *   (B) i = a-1, j = b-1, a < b with D(t_a, t_b) < e_{b-1}   (b = n is t_0).
 * 2.5-opt (reading R19): delta_1 = [g_{i+1} + D(t_{i+1},t_j)] + [D(t_{i+1},t_{j+1}) - e_j]
 * and delta_2 = [g_j + D(t_j,t_{i+1})] + [D(t_i,t_j) - e_i], so add
 *   (C) i = p-1, j = q >= p+1  with D(t_p, t_q) < -g_p, and
 *   (D) i = p-1, j = q, 1 <= p <= q-1 with D(t_q, t_p) < -g_q.
 * Every candidate gets its exact delta(s); the result is the minimum over the
 * candidates with delta < 0 of the same key as the plain sweep -- (delta, Fig. 3
 * cell) for best improvement (reading R5), the cell alone for first improvement
 * (reading R20), (delta, cell, type) for 2.5-opt (R19) -- else (0, 1, 0): the
 * plain sweep's answer when no pair improves (reading R7).  A pair found twice
 * is harmless (the minimum is idempotent).
 *
 * "All cities within distance < r of a point" is a plain scan of the cells of
 * a uniform grid that intersect the square [x-r, x+r] x [y-r, y+r]
 * (D < r implies |dx|, |dy| <= sqrt(s) < r + 1/2), testing the exact
 * oracle_dist of every city found there.
 * ------------------------------------------------------------------------- */
typedef struct {
    int64_t G, w;          /* G x G cells of width w */
    int64_t *start;        /* cell c holds city[start[c] .. start[c+1]) */
    int32_t *city;
} oracle_grid;

static void grid_build(oracle_grid *g, const int32_t *xy, int64_t n)
{
    int64_t G = (int64_t)sqrt((double)n / 2.0);
    if (G < 1) G = 1;
    g->G = G;
    g->w = (32768 + G - 1) / G;
    g->start = (int64_t *)calloc(G * G + 1, sizeof(int64_t));
    g->city = (int32_t *)malloc(sizeof(int32_t) * (n > 0 ? n : 1));
    for (int64_t c = 0; c < n; c++) g->start[(xy[2 * c + 1] / g->w) * G + xy[2 * c] / g->w + 1]++;
    for (int64_t k = 0; k < G * G; k++) g->start[k + 1] += g->start[k];
    int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (G * G + 1));
    memcpy(fill, g->start, sizeof(int64_t) * (G * G + 1));
    for (int64_t c = 0; c < n; c++) g->city[fill[(xy[2 * c + 1] / g->w) * G + xy[2 * c] / g->w]++] = (int32_t)c;
    free(fill);
}

static void grid_free(oracle_grid *g)
{
    free(g->start);
    free(g->city);
}

/* Appends to out[] every city c with oracle_dist((x, y), c) < r; returns the count.
 * out must hold n entries. */
static int64_t grid_within(const oracle_grid *g, const int32_t *xy, int64_t x, int64_t y, int64_t r, int32_t *out)
{
    int64_t m = 0;
    if (r <= 0) return 0;
    int64_t cx0 = x - r < 0 ? 0 : (x - r) / g->w, cx1 = (x + r) / g->w;
    int64_t cy0 = y - r < 0 ? 0 : (y - r) / g->w, cy1 = (y + r) / g->w;
    if (cx1 > g->G - 1) cx1 = g->G - 1;
    if (cy1 > g->G - 1) cy1 = g->G - 1;
    for (int64_t cy = cy0; cy <= cy1; cy++)
        for (int64_t cx = cx0; cx <= cx1; cx++)
            for (int64_t k = g->start[cy * g->G + cx]; k < g->start[cy * g->G + cx + 1]; k++) {
                const int32_t c = g->city[k];
                if (oracle_dist(x, y, xy[2 * c], xy[2 * c + 1]) < r) out[m++] = c;
            }
    return m;
}

/* the running minimum of one thread: (delta, cell, type), or the cell alone (first improvement) */
typedef struct {
    int64_t d, i, j, t;
} radius_best;

static void radius_offer(radius_best *b, int first, int64_t d, int64_t i, int64_t j, int64_t t)
{
    if (d >= 0) return; /* only improving moves compete; none -> (0, 1, 0) */
    const int64_t k = oracle_cell(i, j), kb = oracle_cell(b->i, b->j);
    int better;
    if (b->d >= 0) better = 1;
    else if (first) better = k < kb;
    else better = d < b->d || (d == b->d && (k < kb || (k == kb && t < b->t)));
    if (better) {
        b->d = d; b->i = i; b->j = j; b->t = t;
    }
}

/* One radius-pruned sweep over the route arrays px/py (n+1 entries, closed),
 * e (edges), g (2.5-opt gains, mode 2 only) and pos (city -> position).
 * mode 0: best-improvement 2-opt; 1: first-improvement 2-opt; 2: 2.5-opt. */
static void radius_sweep(const int32_t *xy, int64_t n, const oracle_grid *grid, const int64_t *px, const int64_t *py,
                         const int64_t *e, const int64_t *g, const int64_t *pos, int mode,
                         int64_t *bi, int64_t *bj, int64_t *btype, int64_t *bdelta)
{
    radius_best best = {0, 0, 1, 0};
#pragma omp parallel
    {
        radius_best tb = {0, 0, 1, 0};
        int32_t *near = (int32_t *)malloc(sizeof(int32_t) * n);
#pragma omp for schedule(dynamic, 64) nowait
        for (int64_t p = 0; p <= n; p++) {
            /* the candidate pairs (i, j) of rules A-D anchored at position p */
            for (int rule = 0; rule < 4; rule++) {
                int64_t r;
                if (rule == 0) r = p <= n - 2 ? e[p] : 0;                  /* A: i = p */
                else if (rule == 1) r = p >= 2 ? e[p - 1] : 0;              /* B: j + 1 = p */
                else if (mode != 2) r = 0;
                else if (rule == 2) r = (p >= 1 && p <= n - 2) ? -g[p] : 0; /* C: i + 1 = p */
                else r = (p >= 2 && p <= n - 1) ? -g[p] : 0;                 /* D: j = p */
                const int64_t m = grid_within(grid, xy, px[p], py[p], r, near);
                for (int64_t k = 0; k < m; k++) {
                    const int64_t q = pos[near[k]];
                    int64_t i, j;
                    if (rule == 0) { if (q <= p) continue; i = p; j = q; }
                    else if (rule == 1) { if (q < 1 || q >= p) continue; i = q - 1; j = p - 1; }
                    else if (rule == 2) { if (q < p + 1) continue; i = p - 1; j = q; }
                    else { if (q < 1 || q > p - 1) continue; i = q - 1; j = p; }
                    const int64_t dij = oracle_dist(px[i], py[i], px[j], py[j]);
                    const int64_t di1j1 = oracle_dist(px[i + 1], py[i + 1], px[j + 1], py[j + 1]);
                    radius_offer(&tb, mode == 1, dij + di1j1 - e[i] - e[j], i, j, 0);
                    if (mode == 2 && j >= i + 2) {
                        const int64_t di1j = oracle_dist(px[i + 1], py[i + 1], px[j], py[j]);
                        radius_offer(&tb, 0, g[i + 1] + di1j + di1j1 - e[j], i, j, 1);
                        radius_offer(&tb, 0, g[j] + dij + di1j - e[i], i, j, 2);
                    }
                }
            }
        }
        free(near);
#pragma omp critical
        {
            if (tb.d < 0) radius_offer(&best, mode == 1, tb.d, tb.i, tb.j, tb.t);
        }
    }
    *bi = best.i; *bj = best.j; *btype = best.t; *bdelta = best.d;
}

/* route arrays of `tour`: P[k] = coords[t[k mod n]] for k <= n, e_k, g_k (R19), pos */
static void radius_route(const int32_t *xy, int64_t n, const int32_t *tour, int64_t *px, int64_t *py, int64_t *e,
                         int64_t *g, int64_t *pos)
{
    for (int64_t k = 0; k <= n; k++) {
        const int64_t c = tour[k % n];
        px[k] = xy[2 * c];
        py[k] = xy[2 * c + 1];
    }
    for (int64_t k = 0; k < n; k++) e[k] = oracle_dist(px[k], py[k], px[k + 1], py[k + 1]);
    for (int64_t k = 0; k < n; k++) {
        const int64_t km = (k + n - 1) % n;
        g[k] = oracle_dist(px[km], py[km], px[k + 1], py[k + 1]) - e[km] - e[k];
    }
    for (int64_t k = 0; k < n; k++) pos[tour[k]] = k;
}

/* One sweep from scratch: (i, j, type, delta), equal to oracle_best_move (mode 0),
 * oracle_first_move (mode 1) or oracle25_best_move (mode 2). */
void oracle_radius_best_move(const int32_t *xy, int64_t n, const int32_t *tour, int mode,
                             int64_t *bi, int64_t *bj, int64_t *btype, int64_t *bdelta)
{
    oracle_grid grid;
    grid_build(&grid, xy, n);
    int64_t *buf = (int64_t *)malloc(sizeof(int64_t) * (5 * n + 2));
    int64_t *px = buf, *py = buf + n + 1, *e = buf + 2 * n + 2, *g = buf + 3 * n + 2, *pos = buf + 4 * n + 2;
    radius_route(xy, n, tour, px, py, e, g, pos);
    radius_sweep(xy, n, &grid, px, py, e, g, pos, mode, bi, bj, btype, bdelta);
    free(buf);
    grid_free(&grid);
}

/* Local search with the radius-pruned sweep: the same loop, status and trace
 * conventions as oracle_local_search / oracle_first_local_search (mode 0 / 1;
 * trace rows (i, j, delta)) and oracle25_local_search (mode 2; rows (i, j,
 * delta, type)).  The grid indexes cities, which never move, so it is built
 * once; the route arrays are rebuilt from the tour before every sweep. */
int oracle_radius_local_search(const int32_t *xy, int64_t n, int32_t *tour, int64_t max_iters, int mode,
                               int64_t *length, int64_t *iterations, int64_t *trace, int64_t trace_cap)
{
    oracle_grid grid;
    grid_build(&grid, xy, n);
    int64_t *buf = (int64_t *)malloc(sizeof(int64_t) * (5 * n + 2));
    int64_t *px = buf, *py = buf + n + 1, *e = buf + 2 * n + 2, *g = buf + 3 * n + 2, *pos = buf + 4 * n + 2;
    const int w = mode == 2 ? 4 : 3;
    int64_t L = oracle_tour_length(xy, n, tour);
    int64_t it = 0;
    int status = 0;
    for (;;) {
        int64_t i, j, t, d;
        radius_route(xy, n, tour, px, py, e, g, pos);
        radius_sweep(xy, n, &grid, px, py, e, g, pos, mode, &i, &j, &t, &d);
        if (d >= 0) break;
        if (max_iters >= 0 && it >= max_iters) { /* reading R8 */
            status = 1;
            break;
        }
        if (mode == 2) oracle25_apply(tour, i, j, (int)t);
        else oracle_apply(tour, i, j);
        L += d;
        if (trace && it < trace_cap) {
            trace[w * it] = i; trace[w * it + 1] = j; trace[w * it + 2] = d;
            if (w == 4) trace[w * it + 3] = t;
        }
        it++;
    }
    free(buf);
    grid_free(&grid);
    *length = L;
    *iterations = it;
    return status;
}
