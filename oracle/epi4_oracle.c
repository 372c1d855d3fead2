/*
 * epi4_oracle.c — plain CPU oracle for the exhaustive fourth-order K2 epistasis search.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code,
 * header, table or constant generator with the CUDA path (paper_conf_icpp_nobreiss22_b200/),
 * and it reads BYTE genotypes, never bit planes.
 *
 * What it computes is the plain definition; the passages followed:
 *   PAPER.md:L47  (§2)   a fourth-order search finds the SNP quad most associated with the
 *                        phenotype; each quad has 81 (3^4) genotypes, counted separately for
 *                        cases and controls -> a 2 x 81 contingency table (162 values).
 *   PAPER.md:L53-59, L143 (§2, §3.5)  Bayesian K2 score, sums of logarithms written as
 *                        log-factorials via Gamma(x) = (x-1)!  (reading #1 in DESIGN.md):
 *                        K2 = sum_{c=0}^{80} [ lgamma(r_c + 2) - lgamma(r_c0 + 1) - lgamma(r_c1 + 1) ],
 *                        r_c = r_c0 + r_c1, natural log.
 *   PAPER.md:L66   (§3.1) genotype codes: 0 = AA, 1 = Aa, 2 = aa.
 *   PAPER.md:L74   (§3.2) a genotype count = number of samples having genotype (a,b,c,d) on the
 *                        four SNPs (AND of 4 indicator vectors + POPC) — here: a per-sample loop.
 *   PAPER.md:L109, L145 (§3.2, §3.5) output = best quad + score; a quad index is packed into 64 bits
 *                        as 4 x 16-bit SNP indices.
 *   PAPER.md:L268  (§4.5) combinations (i<j<k<l), not permutations.
 * Readings fixed by DESIGN.md: #2 best = argmin K2; #3 ties -> the
 * lexicographically smallest quad (= smallest packed index); #4 K2 accumulated in double in
 * canonical cell order c = 27a + 9b + 3c + d, t = (L(r+1) - L(r0)) - L(r1), K2 += t, with
 * L(n) = lgamma(n + 1.0) from glibc; #14 top-k = the k smallest (K2, index) keys, ascending.
 *
 * Pins (tests/test_oracle.py): hand-enumerated dataset (K2 = log 576), closed forms, cell sums
 * equal n0/n1, 4-way -> 3-way/2-way marginalisation vs a separately written numpy brute force,
 * planted-interaction recovery, brute-force top-k on tiny inputs, duplicated-SNP exact ties.
 */
#define _GNU_SOURCE
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define NCELL 81

/* L(n) = log(n!) = lgamma(n + 1)  (Gamma(x) = (x-1)!) */
static double log_factorial(uint32_t n) {
    int sign;
    return lgamma_r((double)n + 1.0, &sign);
}

/* K2 of one 2 x 81 table, r[0..80] = controls, r[81..161] = cases (reading #1/#4). */
double oracle_k2(const uint32_t *r) {
    double k2 = 0.0;
    for (int c = 0; c < NCELL; ++c) {
        uint32_t r0 = r[c], r1 = r[NCELL + c];
        double t = (log_factorial(r0 + r1 + 1) - log_factorial(r0)) - log_factorial(r1);
        k2 = k2 + t;
    }
    return k2;
}

/* packed quad index: i<<48 | j<<32 | k<<16 | l */
uint64_t oracle_pack(int32_t i, int32_t j, int32_t k, int32_t l) {
    return ((uint64_t)(uint16_t)i << 48) | ((uint64_t)(uint16_t)j << 32) |
           ((uint64_t)(uint16_t)k << 16) | (uint64_t)(uint16_t)l;
}

/* 2 x 81 table of one quad by a per-sample loop.
 * geno: N x M SNP-major bytes, phen: M bytes (0 control / 1 case). */
static void count_quad(const uint8_t *geno, const uint8_t *phen, int64_t m,
                       int32_t i, int32_t j, int32_t k, int32_t l, uint32_t *r) {
    const uint8_t *gi = geno + (int64_t)i * m, *gj = geno + (int64_t)j * m;
    const uint8_t *gk = geno + (int64_t)k * m, *gl = geno + (int64_t)l * m;
    memset(r, 0, sizeof(uint32_t) * 2 * NCELL);
    for (int64_t s = 0; s < m; ++s) {
        int cell = 27 * gi[s] + 9 * gj[s] + 3 * gk[s] + gl[s];
        r[phen[s] * NCELL + cell] += 1;
    }
}

static int validate(const uint8_t *geno, const uint8_t *phen, int32_t n, int64_t m) {
    if (n < 3 || n > 65536 || m < 1) return -1;
    for (int64_t s = 0; s < m; ++s) if (phen[s] > 1) return -2;
    for (int64_t x = 0; x < (int64_t)n * m; ++x) if (geno[x] > 2) return -3;
    return 0;
}

/* Tables for an explicit list of quads (any order of the 4 indices is accepted and used as given:
 * cell = 27 g[q0] + 9 g[q1] + 3 g[q2] + g[q3]).  counts: nq x 2 x 81. */
int oracle_tables(const uint8_t *geno, const uint8_t *phen, int32_t n, int64_t m,
                  const int32_t *quads, int64_t nq, uint32_t *counts, int32_t n_threads) {
    int rc = validate(geno, phen, n, m);
    if (rc) return rc;
    for (int64_t q = 0; q < nq; ++q)
        for (int t = 0; t < 4; ++t)
            if (quads[4 * q + t] < 0 || quads[4 * q + t] >= n) return -4;
#ifdef _OPENMP
    if (n_threads > 0) omp_set_num_threads(n_threads);
#pragma omp parallel for schedule(dynamic, 16)
#endif
    for (int64_t q = 0; q < nq; ++q)
        count_quad(geno, phen, m, quads[4 * q], quads[4 * q + 1], quads[4 * q + 2], quads[4 * q + 3],
                   counts + q * 2 * NCELL);
    return 0;
}

/* K2 for an explicit list of quads. */
int oracle_score(const uint8_t *geno, const uint8_t *phen, int32_t n, int64_t m,
                 const int32_t *quads, int64_t nq, double *k2_out, int32_t n_threads) {
    int rc = validate(geno, phen, n, m);
    if (rc) return rc;
#ifdef _OPENMP
    if (n_threads > 0) omp_set_num_threads(n_threads);
#pragma omp parallel for schedule(dynamic, 16)
#endif
    for (int64_t q = 0; q < nq; ++q) {
        uint32_t r[2 * NCELL];
        count_quad(geno, phen, m, quads[4 * q], quads[4 * q + 1], quads[4 * q + 2], quads[4 * q + 3], r);
        k2_out[q] = oracle_k2(r);
    }
    return 0;
}

/* key order: (K2, packed index) lexicographic (readings #2, #3) */
static int key_less(double ka, uint64_t ia, double kb, uint64_t ib) {
    return ka < kb || (ka == kb && ia < ib);
}

/* insert into a sorted list of capacity cap holding *len entries */
static void topk_insert(double *k2, uint64_t *idx, int32_t *len, int32_t cap, double kv, uint64_t iv) {
    int32_t n = *len;
    if (n == cap && !key_less(kv, iv, k2[n - 1], idx[n - 1])) return;
    int32_t p = (n < cap) ? n : cap - 1;
    while (p > 0 && key_less(kv, iv, k2[p - 1], idx[p - 1])) {
        k2[p] = k2[p - 1];
        idx[p] = idx[p - 1];
        --p;
    }
    k2[p] = kv;
    idx[p] = iv;
    if (n < cap) *len = n + 1;
}

/* Exhaustive search over every quad i<j<k<l of SNPs [0, n).
 * Returns the top_k smallest (K2, packed index) keys, ascending; *n_out = min(top_k, C(n,4)). */
int oracle_search(const uint8_t *geno, const uint8_t *phen, int32_t n, int64_t m, int32_t top_k,
                  uint64_t *idx_out, double *k2_out, int32_t *n_out, int32_t n_threads) {
    int rc = validate(geno, phen, n, m);
    if (rc) return rc;
    if (top_k < 1) return -5;
    int64_t npairs = (int64_t)n * (n - 1) / 2;
    int32_t nthr = 1;
#ifdef _OPENMP
    if (n_threads > 0) omp_set_num_threads(n_threads);
    nthr = omp_get_max_threads();
#endif
    double *tk = (double *)malloc(sizeof(double) * (size_t)top_k * nthr);
    uint64_t *ti = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)top_k * nthr);
    int32_t *tl = (int32_t *)calloc(nthr, sizeof(int32_t));
    if (!tk || !ti || !tl) { free(tk); free(ti); free(tl); return -6; }
#ifdef _OPENMP
#pragma omp parallel
#endif
    {
        int32_t tid = 0;
#ifdef _OPENMP
        tid = omp_get_thread_num();
#endif
        double *mk = tk + (size_t)tid * top_k;
        uint64_t *mi = ti + (size_t)tid * top_k;
        uint32_t r[2 * NCELL];
#ifdef _OPENMP
#pragma omp for schedule(dynamic, 1)
#endif
        for (int64_t p = 0; p < npairs; ++p) {
            /* p -> (i, j), i < j, lexicographic */
            int32_t i = 0;
            int64_t rem = p;
            while (rem >= n - 1 - i) { rem -= n - 1 - i; ++i; }
            int32_t j = i + 1 + (int32_t)rem;
            for (int32_t k = j + 1; k < n; ++k)
                for (int32_t l = k + 1; l < n; ++l) {
                    count_quad(geno, phen, m, i, j, k, l, r);
                    topk_insert(mk, mi, &tl[tid], top_k, oracle_k2(r), oracle_pack(i, j, k, l));
                }
        }
    }
    /* deterministic merge of the per-thread lists */
    int32_t len = 0;
    double *fk = (double *)malloc(sizeof(double) * top_k);
    uint64_t *fi = (uint64_t *)malloc(sizeof(uint64_t) * top_k);
    for (int32_t t = 0; t < nthr; ++t)
        for (int32_t e = 0; e < tl[t]; ++e)
            topk_insert(fk, fi, &len, top_k, tk[(size_t)t * top_k + e], ti[(size_t)t * top_k + e]);
    memcpy(k2_out, fk, sizeof(double) * len);
    memcpy(idx_out, fi, sizeof(uint64_t) * len);
    *n_out = len;
    free(fk); free(fi); free(tk); free(ti); free(tl);
    return 0;
}

/* ---- alternative objective (the table does not depend on the
 * score): mutual information between the 81-cell genotype of the quad and the phenotype, by its definition
 * I = sum_{c,p} (r_cp / M) ln(r_cp M / (r_c n_p)), written as M*I = sum_c [(X(r_c0) + X(r_c1)) - X(r_c)]
 * + (X(M) - X(n0) - X(n1)) with X(k) = k ln k, X(0) = 0 (0 ln 0 = 0), in canonical cell order.  Ranked
 * largest first: the key is -M*I, ties by the smallest packed index. */
static double xlogx(uint32_t k) { return k ? (double)k * log((double)k) : 0.0; }
double oracle_mi(const uint32_t *r) {   /* M * I of one 2 x 81 table */
    uint32_t n0 = 0, n1 = 0;
    for (int c = 0; c < NCELL; ++c) { n0 += r[c]; n1 += r[NCELL + c]; }
    double acc = 0.0;
    for (int c = 0; c < NCELL; ++c) {
        uint32_t r0 = r[c], r1 = r[NCELL + c];
        acc = acc + ((xlogx(r0) + xlogx(r1)) - xlogx(r0 + r1));
    }
    const double M = (double)(n0 + n1);
    const double cst = (M > 0 ? M * log(M) : 0.0) - xlogx(n0) - xlogx(n1);
    return acc + cst;
}

int oracle_search_mi(const uint8_t *geno, const uint8_t *phen, int32_t n, int64_t m, int32_t top_k,
                     uint64_t *idx_out, double *key_out, int32_t *n_out) {
    int rc = validate(geno, phen, n, m);
    if (rc) return rc;
    if (top_k < 1) return -5;
    int32_t len = 0;
    uint32_t r[2 * NCELL];
    for (int32_t i = 0; i < n; ++i)
        for (int32_t j = i + 1; j < n; ++j)
            for (int32_t k = j + 1; k < n; ++k)
                for (int32_t l = k + 1; l < n; ++l) {
                    count_quad(geno, phen, m, i, j, k, l, r);
                    topk_insert(key_out, idx_out, &len, top_k, -oracle_mi(r), oracle_pack(i, j, k, l));
                }
    *n_out = len;
    return 0;
}

/* ---- second alternative objective ("e.g. mutual information, chi^2"): Pearson's
 * chi-square statistic of the 2 x 81 (phenotype x genotype cell) table, no continuity correction, over the
 * cells with r_c = r_c0 + r_c1 > 0 (an empty genotype column has no expected count and is dropped, the usual
 * contingency-table convention):  X^2 = sum_{c: r_c > 0} sum_p (r_cp - E_cp)^2 / E_cp,  E_cp = r_c n_p / M.
 * Expanding the square, sum_p (r_cp - E_cp)^2 / E_cp = (M / r_c) sum_p r_cp^2 / n_p - r_c, so
 *     X^2 = M * S / (n0 n1) - M,   S = sum_{c: r_c > 0} (r_c0^2 n1 + r_c1^2 n0) / r_c,
 * with the numerator an exact integer (< n0 n1 M < 2^53 whenever the counts pack into 32 bits with room; the
 * GPU library checks the bound) and one correctly rounded division per cell, summed in canonical cell order.
 * X^2 := 0 when a phenotype is empty (no variation).  Ranked largest first: key = -X^2, ties by the smallest
 * packed index.  Pinned in tests/test_oracle3.py against scipy.stats.chi2_contingency (correction=False) and
 * closed forms (independence -> 0; perfect association -> M). */
double oracle_chi2(const uint32_t *r) {   /* X^2 of one 2 x 81 table */
    uint32_t n0 = 0, n1 = 0;
    for (int c = 0; c < NCELL; ++c) { n0 += r[c]; n1 += r[NCELL + c]; }
    if (n0 == 0 || n1 == 0) return 0.0;
    double s = 0.0;
    for (int c = 0; c < NCELL; ++c) {
        const uint64_t r0 = r[c], r1 = r[NCELL + c], rc = r0 + r1;
        if (rc == 0) continue;
        const uint64_t num = r0 * r0 * n1 + r1 * r1 * n0;
        s = s + (double)num / (double)rc;
    }
    const double M = (double)n0 + (double)n1;
    return (M * s) / ((double)n0 * (double)n1) - M;
}

int oracle_search_chi2(const uint8_t *geno, const uint8_t *phen, int32_t n, int64_t m, int32_t top_k,
                       uint64_t *idx_out, double *key_out, int32_t *n_out) {
    int rc = validate(geno, phen, n, m);
    if (rc) return rc;
    if (top_k < 1) return -5;
    int32_t len = 0;
    uint32_t r[2 * NCELL];
    for (int32_t i = 0; i < n; ++i)
        for (int32_t j = i + 1; j < n; ++j)
            for (int32_t k = j + 1; k < n; ++k)
                for (int32_t l = k + 1; l < n; ++l) {
                    count_quad(geno, phen, m, i, j, k, l, r);
                    topk_insert(key_out, idx_out, &len, top_k, -oracle_chi2(r), oracle_pack(i, j, k, l));
                }
    *n_out = len;
    return 0;
}

/* ---- third-order search (the paper's predecessors) ----------
 * The same definition one order lower: every triple i<j<k, its 2 x 27 genotype table by a per-sample loop
 * (cell = 9 g_i + 3 g_j + g_k), K2 = sum_{c=0}^{26} [(L(r_c + 1) - L(r_c0)) - L(r_c1)] in canonical cell order,
 * top-k smallest (K2, index) keys with index = i<<48 | j<<32 | k<<16 (the quad packing with l = 0). */
#define NCELL3 27
static void count_triple(const uint8_t *geno, const uint8_t *phen, int64_t m, int32_t i, int32_t j, int32_t k,
                         uint32_t *r) {
    const uint8_t *gi = geno + (int64_t)i * m, *gj = geno + (int64_t)j * m, *gk = geno + (int64_t)k * m;
    memset(r, 0, sizeof(uint32_t) * 2 * NCELL3);
    for (int64_t s = 0; s < m; ++s) r[phen[s] * NCELL3 + 9 * gi[s] + 3 * gj[s] + gk[s]] += 1;
}
static double k2_27(const uint32_t *r) {
    double k2 = 0.0;
    for (int c = 0; c < NCELL3; ++c) {
        uint32_t r0 = r[c], r1 = r[NCELL3 + c];
        double t = (log_factorial(r0 + r1 + 1) - log_factorial(r0)) - log_factorial(r1);
        k2 = k2 + t;
    }
    return k2;
}

/* 2 x 27 tables of an explicit triple list (indices used as given). counts: nt x 2 x 27 */
int oracle_tables3(const uint8_t *geno, const uint8_t *phen, int32_t n, int64_t m, const int32_t *tri, int64_t nt,
                   uint32_t *counts) {
    int rc = validate(geno, phen, n, m);
    if (rc) return rc;
    for (int64_t t = 0; t < nt; ++t) {
        for (int u = 0; u < 3; ++u)
            if (tri[3 * t + u] < 0 || tri[3 * t + u] >= n) return -4;
        count_triple(geno, phen, m, tri[3 * t], tri[3 * t + 1], tri[3 * t + 2], counts + t * 2 * NCELL3);
    }
    return 0;
}

int oracle_search3(const uint8_t *geno, const uint8_t *phen, int32_t n, int64_t m, int32_t top_k,
                   uint64_t *idx_out, double *k2_out, int32_t *n_out, int32_t n_threads) {
    int rc = validate(geno, phen, n, m);
    if (rc) return rc;
    if (top_k < 1) return -5;
    int32_t nthr = 1;
#ifdef _OPENMP
    if (n_threads > 0) omp_set_num_threads(n_threads);
    nthr = omp_get_max_threads();
#endif
    double *tk = (double *)malloc(sizeof(double) * (size_t)top_k * nthr);
    uint64_t *ti = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)top_k * nthr);
    int32_t *tl = (int32_t *)calloc(nthr, sizeof(int32_t));
    if (!tk || !ti || !tl) { free(tk); free(ti); free(tl); return -6; }
#ifdef _OPENMP
#pragma omp parallel
#endif
    {
        int32_t tid = 0;
#ifdef _OPENMP
        tid = omp_get_thread_num();
#endif
        uint32_t r[2 * NCELL3];
#ifdef _OPENMP
#pragma omp for schedule(dynamic, 1)
#endif
        for (int32_t i = 0; i < n; ++i)
            for (int32_t j = i + 1; j < n; ++j)
                for (int32_t k = j + 1; k < n; ++k) {
                    count_triple(geno, phen, m, i, j, k, r);
                    topk_insert(tk + (size_t)tid * top_k, ti + (size_t)tid * top_k, &tl[tid], top_k, k2_27(r),
                                oracle_pack(i, j, k, 0));
                }
    }
    int32_t len = 0;
    double *fk = (double *)malloc(sizeof(double) * top_k);
    uint64_t *fi = (uint64_t *)malloc(sizeof(uint64_t) * top_k);
    for (int32_t t = 0; t < nthr; ++t)
        for (int32_t e = 0; e < tl[t]; ++e)
            topk_insert(fk, fi, &len, top_k, tk[(size_t)t * top_k + e], ti[(size_t)t * top_k + e]);
    memcpy(k2_out, fk, sizeof(double) * len);
    memcpy(idx_out, fi, sizeof(uint64_t) * len);
    *n_out = len;
    free(fk); free(fi); free(tk); free(ti); free(tl);
    return 0;
}

/* threads the OpenMP runtime will use (for the cpu_baseline "cores" field) */
int32_t oracle_max_threads(int32_t n_threads) {
#ifdef _OPENMP
    if (n_threads > 0) omp_set_num_threads(n_threads);
    return omp_get_max_threads();
#else
    (void)n_threads;
    return 1;
#endif
}

/* ---- third-order search with the alternative objectives (SURVEY.md §8(f) NEXT-3 x NEXT-4) ---------------
 * The same definitions as oracle_mi / oracle_chi2 on the 2 x 27 table of a triple (cell 9a + 3b + c), in
 * canonical cell order: objective 1 = mutual information (key -M*I), 2 = Pearson chi-square (key -X^2);
 * top-k smallest (key, index) with index = i<<48 | j<<32 | k<<16.  Single-threaded (small test problems). */
static double mi_27(const uint32_t *r) {
    uint32_t n0 = 0, n1 = 0;
    for (int c = 0; c < NCELL3; ++c) { n0 += r[c]; n1 += r[NCELL3 + c]; }
    double acc = 0.0;
    for (int c = 0; c < NCELL3; ++c) {
        uint32_t r0 = r[c], r1 = r[NCELL3 + c];
        acc = acc + ((xlogx(r0) + xlogx(r1)) - xlogx(r0 + r1));
    }
    const double M = (double)(n0 + n1);
    const double cst = (M > 0 ? M * log(M) : 0.0) - xlogx(n0) - xlogx(n1);
    return acc + cst;
}
static double chi2_27(const uint32_t *r) {
    uint32_t n0 = 0, n1 = 0;
    for (int c = 0; c < NCELL3; ++c) { n0 += r[c]; n1 += r[NCELL3 + c]; }
    if (n0 == 0 || n1 == 0) return 0.0;
    double s = 0.0;
    for (int c = 0; c < NCELL3; ++c) {
        const uint64_t r0 = r[c], r1 = r[NCELL3 + c], rc = r0 + r1;
        if (rc == 0) continue;
        const uint64_t num = r0 * r0 * n1 + r1 * r1 * n0;
        s = s + (double)num / (double)rc;
    }
    const double M = (double)n0 + (double)n1;
    return (M * s) / ((double)n0 * (double)n1) - M;
}
double oracle_score3_obj(const uint32_t *r, int32_t objective) {
    return objective == 1 ? mi_27(r) : objective == 2 ? chi2_27(r) : k2_27(r);
}
int oracle_search3_obj(const uint8_t *geno, const uint8_t *phen, int32_t n, int64_t m, int32_t top_k,
                       int32_t objective, uint64_t *idx_out, double *key_out, int32_t *n_out) {
    int rc = validate(geno, phen, n, m);
    if (rc) return rc;
    if (top_k < 1 || objective < 1 || objective > 2) return -5;
    int32_t len = 0;
    uint32_t r[2 * NCELL3];
    for (int32_t i = 0; i < n; ++i)
        for (int32_t j = i + 1; j < n; ++j)
            for (int32_t k = j + 1; k < n; ++k) {
                count_triple(geno, phen, m, i, j, k, r);
                topk_insert(key_out, idx_out, &len, top_k, -oracle_score3_obj(r, objective), oracle_pack(i, j, k, 0));
            }
    *n_out = len;
    return 0;
}
