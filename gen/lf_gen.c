/*
 * lf_gen.c -- seeded, counter-based synthetic sparse-matrix and dense-value
 * generators.  Shared by BOTH sides (the oracle/ tests and the CUDA path's
 * tests + bench): it holds none of the method's arithmetic (no bucketing, no
 * cost model, no SpMM) -- only the inputs' shapes.
 *
 * Every random number is a pure function of (seed, stream, index):
 *     lfgen_u64(seed, stream, idx) = mix(mix(mix(seed) ^ stream) ^ idx)
 * with mix = the splitmix64 finaliser.  OpenMP loops are therefore
 * deterministic regardless of the thread count.
 *
 * Workload shapes follow the paper's datasets (Table 4)
 * and SURVEY.md section 8(d):
 *   - uniform Erdos-Renyi            (config 1)
 *   - R-MAT / Graph500 power law     (config 2)
 *   - 27-point stencil (banded FEM)  (config 3)
 *   - lognormal-degree Chung-Lu graph shaped like reddit (config 4)
 *   - full band of half-width hw     (mixed-skew suite)
 * Output: CSR with int64 row_ptr, int32 col_ind, columns sorted ascending per
 * row (duplicates removed unless stated).  Values are filled separately by
 * lfgen_fill_values().
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif

enum {
    LFGEN_STREAM_RMAT = 0x524d4154u,
    LFGEN_STREAM_PERM = 0x5045524du,
    LFGEN_STREAM_ER = 0x45520000u,
    LFGEN_STREAM_DEG = 0x44454700u,
    LFGEN_STREAM_CPERM = 0x43504552u,
    LFGEN_STREAM_COL = 0x434f4c00u,
};

static inline uint64_t mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

uint64_t lfgen_u64(uint64_t seed, uint64_t stream, uint64_t idx) {
    return mix64(mix64(mix64(seed) ^ stream) ^ idx);
}

/* uniform double in the open interval (0,1) */
static inline double u01(uint64_t u) { return ((double)(u >> 11) + 0.5) * (1.0 / 9007199254740992.0); }

typedef struct {
    int64_t n_rows, n_cols, nnz;
    int64_t *row_ptr; /* [n_rows+1] */
    int32_t *col_ind; /* [nnz] */
} lfgen_csr;

void lfgen_free(lfgen_csr *m) {
    if (!m) return;
    free(m->row_ptr);
    free(m->col_ind);
    m->row_ptr = NULL;
    m->col_ind = NULL;
}

static int cmp_i32(const void *a, const void *b) {
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

static void sort_i32(int32_t *v, int64_t n) {
    if (n < 32) { /* insertion sort */
        for (int64_t i = 1; i < n; i++) {
            int32_t x = v[i];
            int64_t j = i - 1;
            while (j >= 0 && v[j] > x) { v[j + 1] = v[j]; j--; }
            v[j + 1] = x;
        }
    } else {
        qsort(v, (size_t)n, sizeof(int32_t), cmp_i32);
    }
}

/* Edge list -> CSR (rows sorted, columns sorted per row, optional dedup). */
static int edges_to_csr(int64_t n_rows, int64_t n_cols, int64_t E, const int32_t *er, const int32_t *ec,
                        int dedup, lfgen_csr *out) {
    int64_t *cnt = (int64_t *)calloc((size_t)n_rows + 1, sizeof(int64_t));
    int32_t *tmp = (int32_t *)malloc((size_t)(E > 0 ? E : 1) * sizeof(int32_t));
    if (!cnt || !tmp) { free(cnt); free(tmp); return -1; }
    for (int64_t e = 0; e < E; e++) cnt[er[e] + 1]++;
    for (int64_t i = 0; i < n_rows; i++) cnt[i + 1] += cnt[i];
    {
        int64_t *cur = (int64_t *)malloc((size_t)(n_rows + 1) * sizeof(int64_t));
        if (!cur) { free(cnt); free(tmp); return -1; }
        memcpy(cur, cnt, (size_t)(n_rows + 1) * sizeof(int64_t));
        for (int64_t e = 0; e < E; e++) tmp[cur[er[e]]++] = ec[e];
        free(cur);
    }
    int64_t *newlen = (int64_t *)malloc((size_t)(n_rows + 1) * sizeof(int64_t));
    if (!newlen) { free(cnt); free(tmp); return -1; }
#pragma omp parallel for schedule(dynamic, 256)
    for (int64_t i = 0; i < n_rows; i++) {
        int32_t *r = tmp + cnt[i];
        int64_t n = cnt[i + 1] - cnt[i];
        sort_i32(r, n);
        int64_t m = n;
        if (dedup && n > 1) {
            m = 1;
            for (int64_t q = 1; q < n; q++)
                if (r[q] != r[m - 1]) r[m++] = r[q];
        }
        newlen[i] = m;
    }
    out->n_rows = n_rows;
    out->n_cols = n_cols;
    out->row_ptr = (int64_t *)malloc((size_t)(n_rows + 1) * sizeof(int64_t));
    if (!out->row_ptr) { free(cnt); free(tmp); free(newlen); return -1; }
    out->row_ptr[0] = 0;
    for (int64_t i = 0; i < n_rows; i++) out->row_ptr[i + 1] = out->row_ptr[i] + newlen[i];
    out->nnz = out->row_ptr[n_rows];
    out->col_ind = (int32_t *)malloc((size_t)(out->nnz > 0 ? out->nnz : 1) * sizeof(int32_t));
    if (!out->col_ind) { free(cnt); free(tmp); free(newlen); free(out->row_ptr); return -1; }
#pragma omp parallel for schedule(dynamic, 256)
    for (int64_t i = 0; i < n_rows; i++)
        memcpy(out->col_ind + out->row_ptr[i], tmp + cnt[i], (size_t)newlen[i] * sizeof(int32_t));
    free(cnt);
    free(tmp);
    free(newlen);
    return 0;
}

/* random permutation of [0,n): sort indices by a hash key (ties impossible in practice,
 * broken by index) */
typedef struct { uint64_t key; int64_t idx; } kv_t;
static int cmp_kv(const void *a, const void *b) {
    const kv_t *x = (const kv_t *)a, *y = (const kv_t *)b;
    if (x->key != y->key) return x->key < y->key ? -1 : 1;
    return (x->idx > y->idx) - (x->idx < y->idx);
}
static int32_t *make_perm(int64_t n, uint64_t seed, uint64_t stream) {
    kv_t *kv = (kv_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(kv_t));
    int32_t *perm = (int32_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int32_t));
    if (!kv || !perm) { free(kv); free(perm); return NULL; }
    for (int64_t i = 0; i < n; i++) { kv[i].key = lfgen_u64(seed, stream, (uint64_t)i); kv[i].idx = i; }
    qsort(kv, (size_t)n, sizeof(kv_t), cmp_kv);
    for (int64_t i = 0; i < n; i++) perm[kv[i].idx] = (int32_t)i;
    free(kv);
    return perm;
}

/* R-MAT (Chakrabarti et al.; Graph500 parameters a,b,c, d=1-a-b-c).  2^scale
 * vertices, edge_factor*2^scale edge draws, rows = source vertex.  One 64-bit
 * draw per (edge, level) picks the quadrant by integer threshold comparison. */
int lfgen_rmat(int32_t scale, int64_t edge_factor, double a, double b, double c, uint64_t seed, int permute,
               int dedup, lfgen_csr *out) {
    memset(out, 0, sizeof(*out));
    if (scale < 1 || scale > 30 || edge_factor < 0) return -2;
    int64_t n = (int64_t)1 << scale;
    int64_t E = edge_factor * n;
    const double two64 = 18446744073709551616.0;
    uint64_t ta = (uint64_t)(a * two64);
    uint64_t tab = (uint64_t)((a + b) * two64);
    uint64_t tabc = (uint64_t)((a + b + c) >= 1.0 ? 18446744073709551615.0 : (a + b + c) * two64);
    int32_t *er = (int32_t *)malloc((size_t)(E > 0 ? E : 1) * sizeof(int32_t));
    int32_t *ec = (int32_t *)malloc((size_t)(E > 0 ? E : 1) * sizeof(int32_t));
    if (!er || !ec) { free(er); free(ec); return -1; }
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < E; e++) {
        uint32_t r = 0, cc = 0;
        for (int l = 0; l < scale; l++) {
            uint64_t u = lfgen_u64(seed, LFGEN_STREAM_RMAT, ((uint64_t)e << 6) | (uint64_t)l);
            uint32_t rb, cb;
            if (u < ta) { rb = 0; cb = 0; }
            else if (u < tab) { rb = 0; cb = 1; }
            else if (u < tabc) { rb = 1; cb = 0; }
            else { rb = 1; cb = 1; }
            r = (r << 1) | rb;
            cc = (cc << 1) | cb;
        }
        er[e] = (int32_t)r;
        ec[e] = (int32_t)cc;
    }
    if (permute) {
        int32_t *perm = make_perm(n, seed, LFGEN_STREAM_PERM);
        if (!perm) { free(er); free(ec); return -1; }
#pragma omp parallel for schedule(static)
        for (int64_t e = 0; e < E; e++) { er[e] = perm[er[e]]; ec[e] = perm[ec[e]]; }
        free(perm);
    }
    int rc = edges_to_csr(n, n, E, er, ec, dedup, out);
    free(er);
    free(ec);
    return rc;
}

/* Erdos-Renyi: each (i,k) present independently with probability p, drawn by
 * geometric skipping along each row (draw index = row*2^32 + draw). */
int lfgen_uniform(int64_t n_rows, int64_t n_cols, double p, uint64_t seed, lfgen_csr *out) {
    memset(out, 0, sizeof(*out));
    if (n_rows < 0 || n_cols < 0 || !(p >= 0.0 && p <= 1.0)) return -2;
    out->n_rows = n_rows;
    out->n_cols = n_cols;
    out->row_ptr = (int64_t *)calloc((size_t)n_rows + 1, sizeof(int64_t));
    if (!out->row_ptr) return -1;
    double lq = (p < 1.0) ? log1p(-p) : 0.0;
    /* pass 1: lengths */
#pragma omp parallel for schedule(dynamic, 256)
    for (int64_t i = 0; i < n_rows; i++) {
        int64_t cnt = 0;
        if (p >= 1.0) cnt = n_cols;
        else if (p > 0.0) {
            int64_t k = -1;
            uint64_t d = 0;
            for (;;) {
                double u = u01(lfgen_u64(seed, LFGEN_STREAM_ER, ((uint64_t)i << 32) | d++));
                k += 1 + (int64_t)floor(log(u) / lq);
                if (k >= n_cols) break;
                cnt++;
            }
        }
        out->row_ptr[i + 1] = cnt;
    }
    for (int64_t i = 0; i < n_rows; i++) out->row_ptr[i + 1] += out->row_ptr[i];
    out->nnz = out->row_ptr[n_rows];
    out->col_ind = (int32_t *)malloc((size_t)(out->nnz > 0 ? out->nnz : 1) * sizeof(int32_t));
    if (!out->col_ind) return -1;
#pragma omp parallel for schedule(dynamic, 256)
    for (int64_t i = 0; i < n_rows; i++) {
        int32_t *dst = out->col_ind + out->row_ptr[i];
        if (p >= 1.0) {
            for (int64_t k = 0; k < n_cols; k++) dst[k] = (int32_t)k;
        } else if (p > 0.0) {
            int64_t k = -1, m = 0;
            uint64_t d = 0;
            for (;;) {
                double u = u01(lfgen_u64(seed, LFGEN_STREAM_ER, ((uint64_t)i << 32) | d++));
                k += 1 + (int64_t)floor(log(u) / lq);
                if (k >= n_cols) break;
                dst[m++] = (int32_t)k;
            }
        }
    }
    return 0;
}

/* 27-point stencil on an n^3 grid, lexicographic order (x fastest); row
 * (z*n+y)*n+x couples to every in-range neighbour with |dz|,|dy|,|dx| <= 1.
 * nnz = (3n-2)^3 exactly. */
int lfgen_stencil27(int64_t n, lfgen_csr *out) {
    memset(out, 0, sizeof(*out));
    if (n < 1 || n * n * n > 2147483647LL) return -2;
    int64_t N = n * n * n;
    out->n_rows = N;
    out->n_cols = N;
    out->row_ptr = (int64_t *)malloc((size_t)(N + 1) * sizeof(int64_t));
    if (!out->row_ptr) return -1;
    out->row_ptr[0] = 0;
    for (int64_t r = 0; r < N; r++) {
        int64_t x = r % n, y = (r / n) % n, z = r / (n * n);
        int64_t cx = 1 + (x > 0) + (x < n - 1), cy = 1 + (y > 0) + (y < n - 1), cz = 1 + (z > 0) + (z < n - 1);
        out->row_ptr[r + 1] = out->row_ptr[r] + cx * cy * cz;
    }
    out->nnz = out->row_ptr[N];
    out->col_ind = (int32_t *)malloc((size_t)out->nnz * sizeof(int32_t));
    if (!out->col_ind) return -1;
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < N; r++) {
        int64_t x = r % n, y = (r / n) % n, z = r / (n * n);
        int64_t q = out->row_ptr[r];
        for (int dz = -1; dz <= 1; dz++) {
            if (z + dz < 0 || z + dz >= n) continue;
            for (int dy = -1; dy <= 1; dy++) {
                if (y + dy < 0 || y + dy >= n) continue;
                for (int dx = -1; dx <= 1; dx++) {
                    if (x + dx < 0 || x + dx >= n) continue;
                    out->col_ind[q++] = (int32_t)(r + dz * n * n + dy * n + dx);
                }
            }
        }
    }
    return 0;
}

/* Full band: row i holds columns max(0,i-hw) .. min(n_cols-1,i+hw). */
int lfgen_banded(int64_t n_rows, int64_t n_cols, int64_t hw, lfgen_csr *out) {
    memset(out, 0, sizeof(*out));
    if (n_rows < 0 || n_cols < 0 || hw < 0) return -2;
    out->n_rows = n_rows;
    out->n_cols = n_cols;
    out->row_ptr = (int64_t *)malloc((size_t)(n_rows + 1) * sizeof(int64_t));
    if (!out->row_ptr) return -1;
    out->row_ptr[0] = 0;
    for (int64_t i = 0; i < n_rows; i++) {
        int64_t lo = i - hw < 0 ? 0 : i - hw, hi = i + hw > n_cols - 1 ? n_cols - 1 : i + hw;
        out->row_ptr[i + 1] = out->row_ptr[i] + (hi >= lo ? hi - lo + 1 : 0);
    }
    out->nnz = out->row_ptr[n_rows];
    out->col_ind = (int32_t *)malloc((size_t)(out->nnz > 0 ? out->nnz : 1) * sizeof(int32_t));
    if (!out->col_ind) return -1;
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n_rows; i++) {
        int64_t lo = i - hw < 0 ? 0 : i - hw;
        for (int64_t q = out->row_ptr[i]; q < out->row_ptr[i + 1]; q++) out->col_ind[q] = (int32_t)(lo + q - out->row_ptr[i]);
    }
    return 0;
}

/* Lognormal-degree Chung-Lu graph (reddit-shaped):
 *   d_i ~ exp(sigma*z_i) rescaled to sum exactly total_nnz, clamped to [1, n];
 *   column weights = a hash-shuffled copy of the degrees;
 *   row i draws d_i DISTINCT columns with probability proportional to the weights
 *   (Vose alias table; duplicates rejected), sorted. */
int lfgen_powerlaw(int64_t n, int64_t total_nnz, double sigma, uint64_t seed, lfgen_csr *out) {
    memset(out, 0, sizeof(*out));
    if (n < 1 || n > 2147483647LL || total_nnz < n || total_nnz > n * n) return -2;
    double *x = (double *)malloc((size_t)n * sizeof(double));
    int64_t *d = (int64_t *)malloc((size_t)n * sizeof(int64_t));
    if (!x || !d) { free(x); free(d); return -1; }
    double sx = 0.0;
    for (int64_t i = 0; i < n; i++) {
        double u1 = u01(lfgen_u64(seed, LFGEN_STREAM_DEG, 2 * (uint64_t)i));
        double u2 = u01(lfgen_u64(seed, LFGEN_STREAM_DEG, 2 * (uint64_t)i + 1));
        double z = sqrt(-2.0 * log(u1)) * cos(6.283185307179586 * u2);
        x[i] = exp(sigma * z);
        sx += x[i];
    }
    double s = (double)total_nnz / sx;
    int64_t sum = 0;
    for (int64_t i = 0; i < n; i++) {
        int64_t v = (int64_t)floor(x[i] * s);
        if (v < 1) v = 1;
        if (v > n) v = n;
        d[i] = v;
        sum += v;
    }
    /* fix the total with deterministic +-1 sweeps in index order */
    while (sum != total_nnz) {
        for (int64_t i = 0; i < n && sum != total_nnz; i++) {
            if (sum < total_nnz && d[i] < n) { d[i]++; sum++; }
            else if (sum > total_nnz && d[i] > 1) { d[i]--; sum--; }
        }
    }
    free(x);
    /* column weights: shuffled degrees */
    int32_t *perm = make_perm(n, seed, LFGEN_STREAM_CPERM);
    double *w = (double *)malloc((size_t)n * sizeof(double));
    double *prob = (double *)malloc((size_t)n * sizeof(double));
    int32_t *alias = (int32_t *)malloc((size_t)n * sizeof(int32_t));
    int32_t *small = (int32_t *)malloc((size_t)n * sizeof(int32_t));
    int32_t *large = (int32_t *)malloc((size_t)n * sizeof(int32_t));
    if (!perm || !w || !prob || !alias || !small || !large) {
        free(d); free(perm); free(w); free(prob); free(alias); free(small); free(large);
        return -1;
    }
    for (int64_t c = 0; c < n; c++) w[perm[c]] = (double)d[c];
    free(perm);
    /* Vose alias */
    double sw = 0.0;
    for (int64_t c = 0; c < n; c++) sw += w[c];
    int64_t ns = 0, nl = 0;
    for (int64_t c = 0; c < n; c++) {
        prob[c] = w[c] * (double)n / sw;
        if (prob[c] < 1.0) small[ns++] = (int32_t)c; else large[nl++] = (int32_t)c;
    }
    while (ns > 0 && nl > 0) {
        int32_t sm = small[--ns], lg = large[--nl];
        alias[sm] = lg;
        prob[lg] = (prob[lg] + prob[sm]) - 1.0;
        if (prob[lg] < 1.0) small[ns++] = lg; else large[nl++] = lg;
    }
    while (nl > 0) { int32_t lg = large[--nl]; prob[lg] = 1.0; alias[lg] = lg; }
    while (ns > 0) { int32_t sm = small[--ns]; prob[sm] = 1.0; alias[sm] = sm; }
    free(small);
    free(large);
    free(w);

    out->n_rows = n;
    out->n_cols = n;
    out->nnz = total_nnz;
    out->row_ptr = (int64_t *)malloc((size_t)(n + 1) * sizeof(int64_t));
    out->col_ind = (int32_t *)malloc((size_t)total_nnz * sizeof(int32_t));
    if (!out->row_ptr || !out->col_ind) { free(d); free(prob); free(alias); return -1; }
    out->row_ptr[0] = 0;
    for (int64_t i = 0; i < n; i++) out->row_ptr[i + 1] = out->row_ptr[i] + d[i];
    int fail = 0;
#pragma omp parallel
    {
        int32_t *stamp = (int32_t *)calloc((size_t)n, sizeof(int32_t));
        if (!stamp) {
#pragma omp atomic write
            fail = 1;
        }
#pragma omp for schedule(dynamic, 64)
        for (int64_t i = 0; i < n; i++) {
            if (!stamp) continue;
            int32_t *dst = out->col_ind + out->row_ptr[i];
            int64_t need = d[i], got = 0;
            uint64_t rs = lfgen_u64(seed, LFGEN_STREAM_COL, (uint64_t)i);
            uint64_t k = 0;
            int32_t tag = (int32_t)(i + 1);
            if (need == n) {
                for (int64_t c = 0; c < n; c++) dst[c] = (int32_t)c;
                continue;
            }
            while (got < need) {
                uint64_t u = mix64(rs ^ mix64(k++));
                int64_t c = (int64_t)(((unsigned __int128)(u >> 11) * (unsigned __int128)n) >> 53);
                double coin = (double)(u & 0x7FFull) * (1.0 / 2048.0) +
                              (double)(mix64(u) >> 11) * (1.0 / 9007199254740992.0) / 2048.0;
                if (coin >= prob[c]) c = alias[c];
                if (stamp[c] != tag) { stamp[c] = tag; dst[got++] = (int32_t)c; }
            }
            sort_i32(dst, need);
        }
        free(stamp);
    }
    free(d);
    free(prob);
    free(alias);
    return fail ? -1 : 0;
}

/* Block-diagonal: dense b x b blocks on the diagonal (n_rows = n_cols = n). */
int lfgen_blockdiag(int64_t n, int64_t b, lfgen_csr *out) {
    memset(out, 0, sizeof(*out));
    if (n < 0 || b < 1) return -2;
    out->n_rows = n;
    out->n_cols = n;
    out->row_ptr = (int64_t *)malloc((size_t)(n + 1) * sizeof(int64_t));
    if (!out->row_ptr) return -1;
    out->row_ptr[0] = 0;
    for (int64_t i = 0; i < n; i++) {
        int64_t lo = i / b * b, hi = lo + b < n ? lo + b : n;
        out->row_ptr[i + 1] = out->row_ptr[i] + (hi - lo);
    }
    out->nnz = out->row_ptr[n];
    out->col_ind = (int32_t *)malloc((size_t)(out->nnz > 0 ? out->nnz : 1) * sizeof(int32_t));
    if (!out->col_ind) return -1;
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; i++) {
        int64_t lo = i / b * b;
        for (int64_t q = out->row_ptr[i]; q < out->row_ptr[i + 1]; q++) out->col_ind[q] = (int32_t)(lo + q - out->row_ptr[i]);
    }
    return 0;
}

/* Arrowhead: the first w rows and the first w columns are dense, plus the
 * diagonal (n_rows = n_cols = n). */
int lfgen_arrowhead(int64_t n, int64_t w, lfgen_csr *out) {
    memset(out, 0, sizeof(*out));
    if (n < 0 || w < 0 || w > n) return -2;
    out->n_rows = n;
    out->n_cols = n;
    out->row_ptr = (int64_t *)malloc((size_t)(n + 1) * sizeof(int64_t));
    if (!out->row_ptr) return -1;
    out->row_ptr[0] = 0;
    for (int64_t i = 0; i < n; i++) out->row_ptr[i + 1] = out->row_ptr[i] + (i < w ? n : w + (i >= w ? 1 : 0));
    out->nnz = out->row_ptr[n];
    out->col_ind = (int32_t *)malloc((size_t)(out->nnz > 0 ? out->nnz : 1) * sizeof(int32_t));
    if (!out->col_ind) return -1;
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; i++) {
        int64_t q = out->row_ptr[i];
        if (i < w) {
            for (int64_t c = 0; c < n; c++) out->col_ind[q++] = (int32_t)c;
        } else {
            for (int64_t c = 0; c < w; c++) out->col_ind[q++] = (int32_t)c;
            out->col_ind[q++] = (int32_t)i;
        }
    }
    return 0;
}

/* Value fills.  kind:
 *   0: on the 2^-23 grid in [-1,1):   (u24 * 2^-23) - 1     (no denormals)
 *   1: integer in [lo,hi]                                   (exact-sum tests)
 *   2: on the 2^-24 grid in [0,1)                           (GNN-style positive)
 *   3: constant 1.0 */
int lfgen_fill_values(float *out, int64_t n, uint64_t seed, uint64_t stream, int32_t kind, int32_t lo, int32_t hi) {
    if (n < 0 || (kind == 1 && hi < lo)) return -2;
#pragma omp parallel for schedule(static)
    for (int64_t q = 0; q < n; q++) {
        uint64_t u = lfgen_u64(seed, stream, (uint64_t)q);
        float v;
        switch (kind) {
        case 0: v = (float)((double)(u >> 40) * (1.0 / 8388608.0) - 1.0); break;
        case 1: v = (float)(lo + (int64_t)(u % (uint64_t)(hi - lo + 1))); break;
        case 2: v = (float)((double)(u >> 40) * (1.0 / 16777216.0)); break;
        default: v = 1.0f; break;
        }
        out[q] = v;
    }
    return 0;
}
