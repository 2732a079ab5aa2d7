/*
 * split_oracle.c — CPU ORACLE for the SPLIT (ICPP'23) GA split search.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_icpp_luoyww0023_b200/, include/split_ga.h)
 * never includes, links or calls anything in oracle/, and this file includes
 * nothing from the product.  Plain C99 + __int128, single-threaded, compiled
 * with -O2 -ffp-contract=off -fno-fast-math so every double operation is one
 * IEEE-754 round-to-nearest operation in source order.
 *
 * Citations: "P@a-b" = characters a..b of PAPER.md (one physical line);
 * readings R1..R16 are listed in DESIGN.md §3.
 *
 * Pins (tests/test_oracle_*.py, all -m "not gpu"):
 *   or_philox4x32_10 .. Random123 known-answer vectors (tests/golden/philox_kat.txt)
 *   or_dexp ........... |error| < 1 ulp vs a 300-bit mpmath exp; dexp(-1) == RN(1/e)
 *   or_fitness ........ closed forms (k=1, two blocks, constant chain), numpy std of the
 *                       explicit block-time list, Eq. 1 identity in exact rationals
 *   or_brute .......... agrees with or_dp (an independent O(k n^2) recursion) on every k
 *   or_count_fixed_k .. C(121,3) = 287,980 (P@9901-10019 with 122 ops, Table 1 P@30163)
 *   or_ga_run ......... invariants (elitism monotone, k range, E=N freeze, pc=pm=0 copies,
 *                       GA best == brute-force optimum on C1, GA best <= DP optimum)
 *                       — the GA trajectory itself is "parity unpinned" by the paper
 *                       (P@21534-22160 gives no operator details; DESIGN.md §3 R7-R11).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include "split_oracle.h"

typedef unsigned __int128 u128;
typedef __int128 i128;

/* ------------------------------------------------------------------------ */
/* Philox4x32-10 — counter-based RNG (Salmon et al., SC'11).  Reading R9:    */
/* the paper only says "randomly chosen" (P@21534-21623); we fix Philox so    */
/* the GA trajectory is reproducible bit for bit.                             */
/* ------------------------------------------------------------------------ */
void or_philox4x32_10(const uint32_t ctr_in[4], const uint32_t key_in[2], uint32_t out[4])
{
    uint32_t c0 = ctr_in[0], c1 = ctr_in[1], c2 = ctr_in[2], c3 = ctr_in[3];
    uint32_t k0 = key_in[0], k1 = key_in[1];
    for (int round = 0; round < 10; ++round) {
        uint64_t p0 = (uint64_t)0xD2511F53u * (uint64_t)c0;
        uint64_t p1 = (uint64_t)0xCD9E8D57u * (uint64_t)c2;
        uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
        uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
        uint32_t n0 = hi1 ^ c1 ^ k0;
        uint32_t n1 = lo1;
        uint32_t n2 = hi0 ^ c3 ^ k1;
        uint32_t n3 = lo0;
        c0 = n0; c1 = n1; c2 = n2; c3 = n3;
        if (round < 9) { k0 += 0x9E3779B9u; k1 += 0xBB67AE85u; }
    }
    out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* draw number d of stream (id, gen, tag) under seed: lane d&3 of block d>>2 */
static uint32_t draw(uint64_t seed, uint32_t id, uint32_t gen, uint32_t tag, uint32_t d)
{
    uint32_t ctr[4] = { id, gen, tag, d >> 2 };
    uint32_t key[2] = { (uint32_t)seed, (uint32_t)(seed >> 32) };
    uint32_t out[4];
    or_philox4x32_10(ctr, key, out);
    return out[d & 3];
}

/* uniform integer in [0, m), m >= 1: floor(u * m / 2^32) (R9, no rejection) */
static uint32_t uniform_below(uint32_t u, uint64_t m) { return (uint32_t)(((uint64_t)u * m) >> 32); }

/* Bernoulli(p): u < floor(p * 2^32) (R9) */
static uint64_t bern_threshold(double p)
{
    if (!(p > 0.0)) return 0;
    if (p >= 1.0) return (uint64_t)1 << 32;
    return (uint64_t)floor(p * 4294967296.0);
}

/* ------------------------------------------------------------------------ */
/* dexp — exp(z) by a fixed operation sequence (reading R5''): Cody-Waite     */
/* reduction by ln 2 and the degree-13 Taylor polynomial with coefficients    */
/* RN(1/i!).  libm exp and CUDA exp are not bit-identical to each other, so   */
/* Eq. 2's e^(...) is pinned to this sequence.                                */
/* ------------------------------------------------------------------------ */
double or_dexp(double z)
{
    static const double INV_LN2 = 0x1.71547652b82fep+0;
    static const double LN2_HI  = 0x1.62e42fefa39efp-1;
    static const double LN2_LO  = 0x1.abc9e3b39803fp-56;
    static const double C[14] = {
        0x1.0000000000000p+0,  0x1.0000000000000p+0,  0x1.0000000000000p-1,
        0x1.5555555555555p-3,  0x1.5555555555555p-5,  0x1.1111111111111p-7,
        0x1.6c16c16c16c17p-10, 0x1.a01a01a01a01ap-13, 0x1.a01a01a01a01ap-16,
        0x1.71de3a556c734p-19, 0x1.27e4fb7789f5cp-22, 0x1.ae64567f544e4p-26,
        0x1.1eed8eff8d898p-29, 0x1.6124613a86d09p-33 };
    if (z > 710.0) return INFINITY;          /* beyond DBL_MAX */
    if (z < -700.0) return 0.0;              /* never reached: Eq. 2 arguments are >= -1 */
    double j = rint(z * INV_LN2);            /* round half to even */
    double r = fma(-j, LN2_HI, z);
    r = fma(-j, LN2_LO, r);
    double p = C[13];
    for (int i = 12; i >= 0; --i) p = fma(p, r, C[i]);
    return ldexp(p, (int)j);
}

/* ------------------------------------------------------------------------ */
/* Fitness, Eq. 2 (P@21101-21296):                                           */
/*   fitness = -( e^(sigma/T - 1) + e^(overhead/m - 1) )                      */
/* Block j of a split runs ops c_{j-1}+1 .. c_j (cuts c_1<...<c_{m-1} at      */
/* operator boundaries, P@8012-8180, P@20780-20831); its time is the sum of   */
/* its operators' profiled latencies (P@18308-18385) plus the overhead of the */
/* cut that starts it (R2, R3).  sigma is the population standard deviation   */
/* of {t_j} (R1: the only convention under which Eq. 1's last equality,       */
/* P@17448-17827, holds), computed exactly as sqrt(m*S2 - S1^2)/m.            */
/* overhead is the ratio OV/T (R4, fn. 2 P@13393-13520).                      */
/* ------------------------------------------------------------------------ */
int or_fitness(uint32_t n, const int64_t* lat, const int64_t* ovh,
               const uint64_t* bits, uint32_t k_min, uint32_t k_max, or_stats* out)
{
    /* T: execution time of the vanilla model (P@21199-21296) */
    int64_t T = 0;
    for (uint32_t i = 0; i < n; ++i) T += lat[i];

    /* cut positions in ascending order; padding bits (p >= n-1) are ignored */
    uint32_t ncut = 0;
    for (uint32_t p = 0; p + 1 < n; ++p)
        if ((bits[p >> 6] >> (p & 63)) & 1u) ++ncut;
    uint32_t k = ncut + 1;                   /* m = number of blocks */
    memset(out, 0, sizeof(*out));
    out->k = k;
    if (k < k_min || k > k_max) { out->fitness = -INFINITY; return 0; }

    /* explicit block times t_1..t_m */
    int64_t* t = (int64_t*)malloc(sizeof(int64_t) * k);
    uint32_t j = 0;
    int64_t cur = 0, OV = 0;
    for (uint32_t i = 0; i < n; ++i) {
        cur += lat[i];
        int cut_here = (i + 1 < n) && ((bits[i >> 6] >> (i & 63)) & 1u);
        if (cut_here || i + 1 == n) {
            t[j++] = cur;
            cur = 0;
            if (cut_here) {                  /* the next block pays this cut's overhead */
                int64_t o = ovh ? ovh[i] : 0;
                cur = o;
                OV += o;
            }
        }
    }
    /* S1 = sum t, S2 = sum t^2, exact */
    i128 S1 = 0, S2 = 0;
    for (j = 0; j < k; ++j) { S1 += t[j]; S2 += (i128)t[j] * t[j]; }
    free(t);
    i128 V = (i128)k * S2 - S1 * S1;         /* = k^2 sigma^2 >= 0 */
    out->s1 = (uint64_t)S1;
    out->s2 = (uint64_t)S2;
    out->overhead = (uint64_t)OV;
    out->var_num = (int64_t)V;
    out->T = (uint64_t)T;

    /* x = sigma/T = sqrt(V)/(k*T);  y = overhead/m = (OV/T)/k   (R5') */
    double x = sqrt((double)(int64_t)V) / ((double)k * (double)T);
    double y = ((double)OV / (double)T) / (double)k;
    double a = or_dexp(x - 1.0);
    double b = or_dexp(y - 1.0);
    out->fitness = -(a + b);
    return 0;
}

double or_fitness_value(uint32_t n, const int64_t* lat, const int64_t* ovh,
                        const uint64_t* bits, uint32_t k_min, uint32_t k_max)
{
    or_stats s;
    or_fitness(n, lat, ovh, bits, k_min, k_max, &s);
    return s.fitness;
}

void or_fitness_batch(uint32_t n, const int64_t* lat, const int64_t* ovh, const uint64_t* bits,
                      uint64_t n_cand, uint32_t k_min, uint32_t k_max, double* f_out)
{
    uint32_t W = (n - 1 + 63) / 64;
    for (uint64_t c = 0; c < n_cand; ++c)
        f_out[c] = or_fitness_value(n, lat, ovh, bits + c * W, k_min, k_max);
}

static void set_bit(uint64_t* row, uint32_t p);

/* ------------------------------------------------------------------------ */
/* Orders.  R10: ranking (f desc, index asc); canonical best (f desc, bitset  */
/* asc as a big-endian unsigned number, word W-1 most significant).           */
/* ------------------------------------------------------------------------ */
static int bits_cmp(const uint64_t* a, const uint64_t* b, uint32_t W)
{
    for (int w = (int)W - 1; w >= 0; --w) {
        if (a[w] < b[w]) return -1;
        if (a[w] > b[w]) return 1;
    }
    return 0;
}

/* 1 if (fa, a) is strictly better than (fb, b) as a best record */
static int record_better(double fa, const uint64_t* a, double fb, const uint64_t* b, uint32_t W)
{
    if (fa > fb) return 1;
    if (fa < fb) return 0;
    return bits_cmp(a, b, W) < 0;
}

/* ------------------------------------------------------------------------ */
/* Exhaustive enumeration of all 2^(n-1) splits (P@9788-10019 shows why the   */
/* paper could not afford it on device: ~1 s of profiling per candidate).     */
/* ------------------------------------------------------------------------ */
int or_brute(uint32_t n, const int64_t* lat, const int64_t* ovh, uint32_t k_min, uint32_t k_max,
             or_brute_result* res, int64_t* minV_per_k /* [n+1] or NULL */,
             uint64_t* argminV_per_k /* [n+1] or NULL */)
{
    if (n < 2 || n > 26) return -1;
    uint64_t total = (uint64_t)1 << (n - 1);
    int have = 0;
    if (minV_per_k) for (uint32_t k = 0; k <= n; ++k) { minV_per_k[k] = -1; if (argminV_per_k) argminV_per_k[k] = 0; }
    for (uint64_t m = 0; m < total; ++m) {
        or_stats s;
        or_fitness(n, lat, ovh, &m, 1, n, &s);
        if (minV_per_k && (minV_per_k[s.k] < 0 || s.var_num < minV_per_k[s.k])) {
            minV_per_k[s.k] = s.var_num;          /* m ascending => first hit is canonical */
            if (argminV_per_k) argminV_per_k[s.k] = m;
        }
        if (s.k < k_min || s.k > k_max) continue;
        if (!have || record_better(s.fitness, &m, res->fitness, &res->bits, 1)) {
            res->fitness = s.fitness;
            res->bits = m;
            res->k = s.k;
            res->var_num = s.var_num;
            have = 1;
        }
    }
    return have ? 0 : -2;
}

/* ------------------------------------------------------------------------ */
/* Exact minimum-variance k-way split by dynamic programming, O(k n^2), for a */
/* constant per-cut overhead delta (R3: ovh[p] = delta):                      */
/*   D[1][i] = P[i]^2,  D[j][i] = min_{p<i} D[j-1][p] + (P[i]-P[p]+delta)^2   */
/* With S1 = T + (k-1) delta fixed, min S2 gives V*_k = k D[k][n] - S1^2.     */
/* ------------------------------------------------------------------------ */
int or_dp(uint32_t n, const int64_t* lat, int64_t delta, uint32_t k_max,
          int64_t* Vstar /* [k_max+1], -1 where infeasible */)
{
    if (n < 1 || k_max < 1) return -1;
    u128* P = (u128*)malloc(sizeof(u128) * (n + 1));
    P[0] = 0;
    for (uint32_t i = 0; i < n; ++i) P[i + 1] = P[i] + (u128)lat[i];
    u128* prev = (u128*)malloc(sizeof(u128) * (n + 1));
    u128* cur = (u128*)malloc(sizeof(u128) * (n + 1));
    const u128 INF = ~(u128)0;
    for (uint32_t i = 0; i <= n; ++i) prev[i] = (i == 0) ? INF : P[i] * P[i];
    for (uint32_t k = 0; k <= k_max; ++k) Vstar[k] = -1;
    u128 T = P[n];
    if (k_max >= 1) Vstar[1] = 0;
    for (uint32_t j = 2; j <= k_max && j <= n; ++j) {
        for (uint32_t i = 0; i <= n; ++i) {
            u128 best = INF;
            for (uint32_t p = j - 1; p < i; ++p) {
                if (prev[p] == INF) continue;
                u128 t = P[i] - P[p] + (u128)delta;
                u128 v = prev[p] + t * t;
                if (v < best) best = v;
            }
            cur[i] = best;
        }
        u128 S1 = T + (u128)(j - 1) * (u128)delta;
        u128 V = (u128)j * cur[n] - S1 * S1;
        Vstar[j] = (int64_t)V;
        u128* tmp = prev; prev = cur; cur = tmp;
    }
    free(P); free(prev); free(cur);
    return 0;
}

/* Fitness of a k-block split with variance numerator V and overhead OV (Eq. 2) */
double or_fitness_from(uint32_t k, int64_t V, int64_t OV, int64_t T)
{
    double x = sqrt((double)V) / ((double)k * (double)T);
    double y = ((double)OV / (double)T) / (double)k;
    return -(or_dexp(x - 1.0) + or_dexp(y - 1.0));
}

/* The two-cut map, synthetic analog of Fig. 2 (P@11560-12128: "The X-axis and
 * Y-axis show position of the first cut point and the second cut point"; (a)
 * splitting overhead, (b) standard deviation of block execution time): for
 * every pair of cut positions a <= b in [0, n-2], the split with cuts {a, b}
 * (3 blocks; a == b is the one-cut split {a}, 2 blocks) scored by or_fitness
 * with no block-count restriction.  Row-major [n-1][n-1] outputs at [a][b];
 * entries a > b get V = -1, OV = 0, fitness = -INFINITY.  Any output may be NULL. */
void or_heatmap2(uint32_t n, const int64_t* lat, const int64_t* ovh, int64_t* var_out, uint64_t* ov_out,
                 double* fit_out)
{
    uint32_t m = n - 1, W = (n - 1 + 63) / 64;
    uint64_t* bits = (uint64_t*)calloc(W, sizeof(uint64_t));
    for (uint32_t a = 0; a < m; ++a)
        for (uint32_t b = 0; b < m; ++b) {
            size_t e = (size_t)a * m + b;
            if (a > b) {
                if (var_out) var_out[e] = -1;
                if (ov_out) ov_out[e] = 0;
                if (fit_out) fit_out[e] = -INFINITY;
                continue;
            }
            memset(bits, 0, sizeof(uint64_t) * W);
            set_bit(bits, a);
            set_bit(bits, b);
            or_stats st;
            or_fitness(n, lat, ovh, bits, 1, n, &st);
            if (var_out) var_out[e] = st.var_num;
            if (ov_out) ov_out[e] = st.overhead;
            if (fit_out) fit_out[e] = st.fitness;
        }
    free(bits);
}

/* Count the fixed-k candidates C(n-1, k-1) by visiting every one (A2). */
uint64_t or_count_fixed_k(uint32_t n, uint32_t k)
{
    uint32_t r = k - 1, m = n - 1;
    if (r > m) return 0;
    if (r == 0) return 1;
    uint32_t* c = (uint32_t*)malloc(sizeof(uint32_t) * r);
    for (uint32_t i = 0; i < r; ++i) c[i] = i;
    uint64_t count = 0;
    for (;;) {
        ++count;
        int i = (int)r - 1;
        while (i >= 0 && c[i] == m - r + (uint32_t)i) --i;
        if (i < 0) break;
        ++c[i];
        for (uint32_t q = (uint32_t)i + 1; q < r; ++q) c[q] = c[q - 1] + 1;
    }
    free(c);
    return count;
}

/* ------------------------------------------------------------------------ */
/* The GA (P@21534-22160), islands run serially.  Step order and every       */
/* operator detail the paper leaves open are fixed by readings R6-R11 in      */
/* DESIGN.md §3 (tags INIT=1 SELECT=2 XOVER=3 MUTATE=4 REPAIR=5).             */
/* ------------------------------------------------------------------------ */
enum { TAG_INIT = 1, TAG_SELECT = 2, TAG_XOVER = 3, TAG_MUTATE = 4, TAG_REPAIR = 5 };

typedef struct {
    uint32_t n, W;
    const int64_t* lat;
    const int64_t* ovh;
    const or_ga_params* p;
    uint64_t seed;
} ga_ctx;

static int get_bit(const uint64_t* row, uint32_t p) { return (int)((row[p >> 6] >> (p & 63)) & 1u); }
static void set_bit(uint64_t* row, uint32_t p) { row[p >> 6] |= (uint64_t)1 << (p & 63); }
static void clr_bit(uint64_t* row, uint32_t p) { row[p >> 6] &= ~((uint64_t)1 << (p & 63)); }
static void flip_bit(uint64_t* row, uint32_t p) { row[p >> 6] ^= (uint64_t)1 << (p & 63); }

static uint32_t count_cuts(const ga_ctx* g, const uint64_t* row)
{
    uint32_t c = 0;
    for (uint32_t p = 0; p + 1 < g->n; ++p) c += (uint32_t)get_bit(row, p);
    return c;
}

/* Step 1 — initial population of randomly chosen cut points (P@21534-21623).
 * k ~ U[k_min, k_max]; k-1 distinct positions from [front_skip, n-2] by
 * Floyd's algorithm ("far from the front", P@19343-19437, via front_skip). */
static void ga_init_row(const ga_ctx* g, uint32_t gid, uint64_t* row)
{
    const or_ga_params* p = g->p;
    memset(row, 0, sizeof(uint64_t) * g->W);
    uint32_t d = 0;
    uint32_t k = p->k_min + uniform_below(draw(g->seed, gid, 0, TAG_INIT, d++), (uint64_t)(p->k_max - p->k_min + 1));
    uint32_t f = p->front_skip;
    uint32_t m = g->n - 1 - f;
    for (uint32_t j = m - (k - 1); j < m; ++j) {
        uint32_t r = uniform_below(draw(g->seed, gid, 0, TAG_INIT, d++), (uint64_t)j + 1);
        if (get_bit(row, f + r)) set_bit(row, f + j);
        else set_bit(row, f + r);
    }
}

/* s-way tournament with replacement (R7): max of (f desc, index asc) */
static uint32_t ga_tournament(const ga_ctx* g, uint32_t gid, uint32_t gen, const double* fit)
{
    uint32_t N = g->p->pop_size;
    uint32_t best = 0;
    for (uint32_t d = 0; d < g->p->tournament_size; ++d) {
        uint32_t idx = uniform_below(draw(g->seed, gid, gen, TAG_SELECT, d), N);
        if (d == 0 || fit[idx] > fit[best] || (fit[idx] == fit[best] && idx < best)) best = idx;
    }
    return best;
}

/* repair (R17): force popcount into [k_min-1, k_max-1] by uniform rank-select */
static void ga_repair(const ga_ctx* g, uint32_t gid, uint32_t gen, uint64_t* row)
{
    uint32_t c = count_cuts(g, row);
    uint32_t d = 0;
    uint32_t npos = g->n - 1;
    while (c > g->p->k_max - 1) {
        uint32_t r = uniform_below(draw(g->seed, gid, gen, TAG_REPAIR, d++), c);
        for (uint32_t pos = 0, seen = 0; pos < npos; ++pos)
            if (get_bit(row, pos)) { if (seen == r) { clr_bit(row, pos); break; } ++seen; }
        --c;
    }
    /* cuts are added only in [front_skip, n-2] (R22: every operator keeps away from
       the front, P@19225-19437); no individual ever has a cut below front_skip */
    uint32_t f = g->p->front_skip;
    while (c < g->p->k_min - 1) {
        uint32_t r = uniform_below(draw(g->seed, gid, gen, TAG_REPAIR, d++), npos - f - c);
        for (uint32_t pos = f, seen = 0; pos < npos; ++pos)
            if (!get_bit(row, pos)) { if (seen == r) { set_bit(row, pos); break; } ++seen; }
        ++c;
    }
}

/* ranking order: (f desc, index asc) */
static const double* g_sort_fit;
static int cmp_rank(const void* a, const void* b)
{
    uint32_t i = *(const uint32_t*)a, j = *(const uint32_t*)b;
    double fi = g_sort_fit[i], fj = g_sort_fit[j];
    if (fi > fj) return -1;
    if (fi < fj) return 1;
    return (i < j) ? -1 : (i > j);
}

typedef struct {
    double f;
    uint32_t src, rank;
    const uint64_t* row;
} migrant;

static int cmp_migrant(const void* a, const void* b)
{
    const migrant* x = (const migrant*)a;
    const migrant* y = (const migrant*)b;
    if (x->f > y->f) return -1;
    if (x->f < y->f) return 1;
    if (x->src != y->src) return x->src < y->src ? -1 : 1;
    return (x->rank < y->rank) ? -1 : (x->rank > y->rank);
}

/* Island migration (reading R16; the island model is the north star's, not
 * the paper's).  Every island exports its top-K by the ranking order (f desc,
 * index asc) -- rows and fitness, snapshotted before any island changes; each
 * island sorts the FOREIGN migrants by (f desc, source island asc, rank asc)
 * and writes the first K into its K worst slots, worst order = (f asc, index
 * desc): the r-th worst slot receives the r-th best migrant.  pop: [I][N][W],
 * fit: [I][N], island i's global id = island_base + i.  1 <= K <= N. */
int or_ga_migrate(uint32_t W, uint32_t N, uint32_t I, uint32_t K, uint32_t island_base,
                  uint64_t* pop, double* fit)
{
    if (I < 2 || K < 1 || K > N) return -1;
    const size_t rowsz = sizeof(uint64_t) * W;
    uint32_t* order = (uint32_t*)malloc(sizeof(uint32_t) * N);
    migrant* all = (migrant*)malloc(sizeof(migrant) * (size_t)I * K);
    uint64_t* snap = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)I * K * W);
    for (uint32_t i = 0; i < I; ++i) {
        for (uint32_t c = 0; c < N; ++c) order[c] = c;
        g_sort_fit = fit + (size_t)i * N;
        qsort(order, N, sizeof(uint32_t), cmp_rank);
        for (uint32_t r = 0; r < K; ++r) {
            migrant* mg = &all[(size_t)i * K + r];
            memcpy(snap + ((size_t)i * K + r) * W, pop + ((size_t)i * N + order[r]) * W, rowsz);
            mg->f = fit[(size_t)i * N + order[r]];
            mg->src = island_base + i;
            mg->rank = r;
            mg->row = snap + ((size_t)i * K + r) * W;
        }
    }
    migrant* foreign = (migrant*)malloc(sizeof(migrant) * (size_t)I * K);
    for (uint32_t i = 0; i < I; ++i) {
        uint32_t nf = 0;
        for (uint32_t s = 0; s < I; ++s)
            if (s != i) for (uint32_t r = 0; r < K; ++r) foreign[nf++] = all[(size_t)s * K + r];
        qsort(foreign, nf, sizeof(migrant), cmp_migrant);
        /* worst order: (f asc, index desc) = reverse of the ranking order */
        for (uint32_t c = 0; c < N; ++c) order[c] = c;
        g_sort_fit = fit + (size_t)i * N;
        qsort(order, N, sizeof(uint32_t), cmp_rank);
        for (uint32_t r = 0; r < K && r < nf; ++r) {
            uint32_t slot = order[N - 1 - r];
            memcpy(pop + ((size_t)i * N + slot) * W, foreign[r].row, rowsz);
            fit[(size_t)i * N + slot] = foreign[r].f;
        }
    }
    free(foreign); free(snap); free(all); free(order);
    return 0;
}

typedef struct {
    double f;
    uint64_t* bits;
    uint32_t gen_found;
    int valid;
} record_t;

static void record_update(const ga_ctx* g, record_t* rec, const uint64_t* pop, const double* fit,
                          uint32_t N, uint32_t gen)
{
    for (uint32_t c = 0; c < N; ++c) {
        const uint64_t* row = pop + (size_t)c * g->W;
        if (!rec->valid || record_better(fit[c], row, rec->f, rec->bits, g->W)) {
            rec->f = fit[c];
            memcpy(rec->bits, row, sizeof(uint64_t) * g->W);
            rec->gen_found = gen;
            rec->valid = 1;
        }
    }
}

int or_ga_run(uint32_t n, const int64_t* lat, const int64_t* ovh, const or_ga_params* p,
              uint32_t generations, uint64_t seed, or_ga_best* best,
              uint64_t* final_pop /* [n_islands][N][W] or NULL */,
              double* final_fit /* [n_islands][N] or NULL */)
{
    ga_ctx g;
    g.n = n; g.W = (n - 1 + 63) / 64; g.lat = lat; g.ovh = ovh; g.p = p; g.seed = seed;
    const uint32_t W = g.W, N = p->pop_size, E = p->n_elite, I = p->n_islands;
    if (n < 2 || N < 2 || E > N || ((N - E) & 1u) || p->tournament_size < 1 || p->tournament_size > 32 ||
        p->k_min < 1 || p->k_min > p->k_max || p->k_max > n || I < 1 ||
        p->k_max - 1 > n - 1 - p->front_skip)
        return -1;
    if (I > 1 && p->migration_interval > 0 && (p->n_migrants < 1 || p->n_migrants > N - E))
        return -1;
    const uint64_t thr_c = bern_threshold(p->p_crossover);
    const uint64_t thr_m = bern_threshold(p->p_mutation);
    const size_t rowsz = sizeof(uint64_t) * W;

    uint64_t* pop = (uint64_t*)calloc((size_t)I * N * W, sizeof(uint64_t));
    uint64_t* nxt = (uint64_t*)calloc((size_t)I * N * W, sizeof(uint64_t));
    double* fit = (double*)calloc((size_t)I * N, sizeof(double));
    double* nfit = (double*)calloc((size_t)I * N, sizeof(double));
    uint32_t* order = (uint32_t*)malloc(sizeof(uint32_t) * N);
    record_t* rec = (record_t*)calloc(I, sizeof(record_t));
    for (uint32_t i = 0; i < I; ++i) rec[i].bits = (uint64_t*)calloc(W, sizeof(uint64_t));
    uint64_t evals = 0;

    /* generation 0 */
    for (uint32_t i = 0; i < I; ++i) {
        for (uint32_t c = 0; c < N; ++c) {
            uint64_t* row = pop + ((size_t)i * N + c) * W;
            ga_init_row(&g, i * N + c, row);
            fit[(size_t)i * N + c] = or_fitness_value(n, lat, ovh, row, p->k_min, p->k_max);
        }
        evals += N;
        record_update(&g, &rec[i], pop + (size_t)i * N * W, fit + (size_t)i * N, N, 0);
    }

    /* global record at the last improvement (R11) */
    uint32_t last_improve = 0;
    double f_improve = -INFINITY;
    for (uint32_t i = 0; i < I; ++i) if (rec[i].f > f_improve) f_improve = rec[i].f;

    uint32_t gen = 0;
    while (gen < generations) {
        for (uint32_t i = 0; i < I; ++i) {
            uint64_t* P0 = pop + (size_t)i * N * W;
            double* F0 = fit + (size_t)i * N;
            uint64_t* P1 = nxt + (size_t)i * N * W;
            double* F1 = nfit + (size_t)i * N;
            /* Step 5 — elites (P@21965-22054): the E best by (f desc, index asc),
             * copied in rank order to slots 0..E-1 of the next generation */
            for (uint32_t c = 0; c < N; ++c) order[c] = c;
            g_sort_fit = F0;
            qsort(order, N, sizeof(uint32_t), cmp_rank);
            for (uint32_t r = 0; r < E; ++r) {
                memcpy(P1 + (size_t)r * W, P0 + (size_t)order[r] * W, rowsz);
                F1[r] = F0[order[r]];
            }
            /* Steps 3-4 — selection, crossover, mutation (P@21745-21963) */
            for (uint32_t c0 = E; c0 < N; c0 += 2) {
                uint32_t c1 = c0 + 1;
                uint32_t gid0 = i * N + c0, gid1 = i * N + c1;
                uint32_t a = ga_tournament(&g, gid0, gen, F0);
                uint32_t b = ga_tournament(&g, gid1, gen, F0);
                uint64_t* ch0 = P1 + (size_t)c0 * W;
                uint64_t* ch1 = P1 + (size_t)c1 * W;
                const uint64_t* A = P0 + (size_t)a * W;
                const uint64_t* B = P0 + (size_t)b * W;
                uint32_t u0 = draw(seed, gid0, gen, TAG_XOVER, 0);
                uint32_t u1 = draw(seed, gid0, gen, TAG_XOVER, 1);
                if ((uint64_t)u0 < thr_c && n >= 3) {
                    /* one-point crossover at x in [1, n-2]: positions < x from the
                     * first parent, positions >= x from the second */
                    uint32_t x = 1 + uniform_below(u1, (uint64_t)(n - 2));
                    memset(ch0, 0, rowsz);
                    memset(ch1, 0, rowsz);
                    for (uint32_t pos = 0; pos + 1 < n; ++pos) {
                        int fa = get_bit(A, pos), fb = get_bit(B, pos);
                        if (pos < x) { if (fa) set_bit(ch0, pos); if (fb) set_bit(ch1, pos); }
                        else         { if (fb) set_bit(ch0, pos); if (fa) set_bit(ch1, pos); }
                    }
                } else {
                    memcpy(ch0, A, rowsz);
                    memcpy(ch1, B, rowsz);
                }
                uint32_t cs[2] = { c0, c1 };
                for (int h = 0; h < 2; ++h) {
                    uint32_t gidh = i * N + cs[h];
                    uint64_t* ch = P1 + (size_t)cs[h] * W;
                    uint32_t m0 = draw(seed, gidh, gen, TAG_MUTATE, 0);
                    uint32_t m1 = draw(seed, gidh, gen, TAG_MUTATE, 1);
                    /* mutation flips a uniform position of [front_skip, n-2] (R22) */
                    if ((uint64_t)m0 < thr_m)
                        flip_bit(ch, p->front_skip + uniform_below(m1, (uint64_t)(n - 1 - p->front_skip)));
                    ga_repair(&g, gidh, gen, ch);
                    /* Step 2 — profile + fitness of the offspring (Eq. 2) */
                    F1[cs[h]] = or_fitness_value(n, lat, ovh, ch, p->k_min, p->k_max);
                }
            }
            evals += N - E;
        }
        { uint64_t* t = pop; pop = nxt; nxt = t; }
        { double* t = fit; fit = nfit; nfit = t; }
        ++gen;
        for (uint32_t i = 0; i < I; ++i)
            record_update(&g, &rec[i], pop + (size_t)i * N * W, fit + (size_t)i * N, N, gen);

        /* Step 6 — termination (P@22056-22160) at sync points (R11) */
        int sync = (I == 1) || (p->migration_interval > 0 && gen % p->migration_interval == 0);
        if (!sync) continue;
        double gf = -INFINITY;
        for (uint32_t i = 0; i < I; ++i) if (rec[i].f > gf) gf = rec[i].f;
        if (gf > f_improve) { f_improve = gf; last_improve = gen; }
        if (p->stall_generations > 0 && gen - last_improve >= p->stall_generations) break;

        /* island migration (R16) */
        if (I > 1 && p->migration_interval > 0 && gen < generations) {
            or_ga_migrate(W, N, I, p->n_migrants, p->island_base, pop, fit);
            for (uint32_t i = 0; i < I; ++i)
                record_update(&g, &rec[i], pop + (size_t)i * N * W, fit + (size_t)i * N, N, gen);
        }
    }

    /* global best: (f desc, bits asc), ties of the same record -> earliest generation */
    uint32_t bi = 0;
    for (uint32_t i = 1; i < I; ++i) {
        if (record_better(rec[i].f, rec[i].bits, rec[bi].f, rec[bi].bits, W)) bi = i;
        else if (rec[i].f == rec[bi].f && bits_cmp(rec[i].bits, rec[bi].bits, W) == 0 &&
                 rec[i].gen_found < rec[bi].gen_found) bi = i;
    }
    or_stats st;
    or_fitness(n, lat, ovh, rec[bi].bits, p->k_min, p->k_max, &st);
    if (best->bits) memcpy(best->bits, rec[bi].bits, rowsz);
    best->fitness = rec[bi].f;
    best->k = st.k;
    best->var_num = st.var_num;
    best->s1 = st.s1;
    best->s2 = st.s2;
    best->overhead = st.overhead;
    best->generation_found = rec[bi].gen_found;
    best->generations_run = gen;
    best->evaluations = evals;
    if (final_pop) memcpy(final_pop, pop, sizeof(uint64_t) * (size_t)I * N * W);
    if (final_fit) memcpy(final_fit, fit, sizeof(double) * (size_t)I * N);

    for (uint32_t i = 0; i < I; ++i) free(rec[i].bits);
    free(rec); free(order); free(pop); free(nxt); free(fit); free(nfit);
    return 0;
}
