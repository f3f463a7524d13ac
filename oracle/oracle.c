/*
 * oracle.c -- SNICIT CPU ORACLE.  TEST INFRASTRUCTURE ONLY (see oracle.h).
 *
 * Plain C, no blocking, no fusion, no reordering beyond what each cited definition states.
 * Build: gcc -O2 -std=c11 -ffp-contract=off -fopenmp -fPIC -shared (see __graft_entry__.build).
 * -ffp-contract=off: every fused multiply-add below is an explicit fmaf()/fma() call.
 *
 * Parity pins for every function: tests/test_oracle_pins.py (brute force, closed forms,
 * Fig. 3b / Fig. 5 worked examples, invariants).  None is "parity unpinned".
 */
#include "oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

int32_t oracle_version(void) { return 1; }

static void set_threads(int32_t nthreads) {
#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#else
    (void)nthreads;
#endif
}

/* sigma(x) = min(max(x, 0), ymax) -- Table 2, PAPER.md:410 ("ReLU with an upper bound of 32",
 * PAPER.md:311-312; ymax = 1 for the medium nets). */
static float sigma_f32(float x, float ymax) { return fminf(fmaxf(x, 0.0f), ymax); }
static double sigma_f64(double x, double ymax) { return fmin(fmax(x, 0.0), ymax); }

/* One layer of Eq. (1) for ONE row, fp32.  target_clones only selects the hardware FMA
 * instruction when the host has one; fmaf() is correctly rounded either way. */
__attribute__((target_clones("fma", "default")))
static void row_layer_f32(int32_t N, const int64_t* p, const int32_t* idx, const float* val,
                          const float* b, float ymax, const float* y, float* y_next) {
    for (int32_t j = 0; j < N; ++j) {
        float acc = 0.0f;
        for (int64_t e = p[j]; e < p[j + 1]; ++e) acc = fmaf(y[idx[e]], val[e], acc);
        y_next[j] = sigma_f32(acc + b[j], ymax);
    }
}

__attribute__((target_clones("fma", "default")))
static void row_layer_f64(int32_t N, const int64_t* p, const int32_t* idx, const float* val,
                          const float* b, double ymax, const double* y, double* y_next) {
    for (int32_t j = 0; j < N; ++j) {
        double acc = 0.0;
        for (int64_t e = p[j]; e < p[j + 1]; ++e) acc = fma(y[idx[e]], (double)val[e], acc);
        y_next[j] = sigma_f64(acc + (double)b[j], ymax);
    }
}

void oracle_layers_f32(int32_t N, const int64_t* ptr, const int32_t* idx, const float* val,
                       const float* bias, float ymax, int32_t l0, int32_t l1,
                       int64_t B, const float* Yin, float* Yout, int32_t nthreads) {
    set_threads(nthreads);
#pragma omp parallel
    {
        float* a = (float*)malloc(sizeof(float) * (size_t)N);
        float* c = (float*)malloc(sizeof(float) * (size_t)N);
#pragma omp for schedule(dynamic, 4)
        for (int64_t r = 0; r < B; ++r) {
            memcpy(a, Yin + r * N, sizeof(float) * (size_t)N);
            for (int32_t l = l0; l < l1; ++l) {
                row_layer_f32(N, ptr + (int64_t)l * (N + 1), idx, val, bias + (int64_t)l * N, ymax, a, c);
                float* tmp = a; a = c; c = tmp;
            }
            memcpy(Yout + r * N, a, sizeof(float) * (size_t)N);
        }
        free(a);
        free(c);
    }
}

void oracle_layers_f64(int32_t N, const int64_t* ptr, const int32_t* idx, const float* val,
                       const float* bias, float ymax, int32_t l0, int32_t l1,
                       int64_t B, const double* Yin, double* Yout, int32_t nthreads) {
    set_threads(nthreads);
#pragma omp parallel
    {
        double* a = (double*)malloc(sizeof(double) * (size_t)N);
        double* c = (double*)malloc(sizeof(double) * (size_t)N);
#pragma omp for schedule(dynamic, 4)
        for (int64_t r = 0; r < B; ++r) {
            memcpy(a, Yin + r * N, sizeof(double) * (size_t)N);
            for (int32_t l = l0; l < l1; ++l) {
                row_layer_f64(N, ptr + (int64_t)l * (N + 1), idx, val, bias + (int64_t)l * N, (double)ymax, a, c);
                double* tmp = a; a = c; c = tmp;
            }
            memcpy(Yout + r * N, a, sizeof(double) * (size_t)N);
        }
        free(a);
        free(c);
    }
}

__attribute__((target_clones("fma", "default")))
static void row_layer_circ_f32(int32_t N, int32_t K, int32_t nu, const float* w, const float* b, float ymax,
                               const float* y, float* y_next) {
    for (int32_t j = 0; j < N; ++j) {
        float acc = 0.0f;
        for (int32_t n = 0; n < K; ++n) {
            int64_t k = (int64_t)j + (int64_t)n * nu; /* (j + n*nu) mod N */
            if (k >= N) k %= N;
            acc = fmaf(y[k], w[n], acc);
        }
        y_next[j] = sigma_f32(acc + b[j], ymax);
    }
}

void oracle_layers_circulant_f32(int32_t N, int32_t K, const int32_t* nu, const float* w, const float* bias,
                                 float ymax, int32_t l0, int32_t l1, int64_t B, const float* Yin, float* Yout,
                                 int32_t nthreads) {
    set_threads(nthreads);
#pragma omp parallel
    {
        float* a = (float*)malloc(sizeof(float) * (size_t)N);
        float* c = (float*)malloc(sizeof(float) * (size_t)N);
#pragma omp for schedule(dynamic, 4)
        for (int64_t r = 0; r < B; ++r) {
            memcpy(a, Yin + r * N, sizeof(float) * (size_t)N);
            for (int32_t l = l0; l < l1; ++l) {
                row_layer_circ_f32(N, K, nu[l], w + (int64_t)l * K, bias + (int64_t)l * N, ymax, a, c);
                float* tmp = a; a = c; c = tmp;
            }
            memcpy(Yout + r * N, a, sizeof(float) * (size_t)N);
        }
        free(a);
        free(c);
    }
}

/* ---- exact fast mode (oracle.h): memoised fixed points of one layer */
static int row_all_equal(const float* y, int32_t N, float v) {
    for (int32_t k = 0; k < N; ++k) if (!(y[k] == v)) return 0;
    return 1;
}

/* fixed[l - l0]: bit 0 = layer l maps the all-zero row to itself, bit 1 = the all-YMAX row to itself,
 * decided by evaluating the layer on those two rows with the plain row function */
static uint8_t* fixed_points(int32_t N, int32_t l0, int32_t l1, float ymax,
                             void (*eval)(int32_t l, const float* y, float* y_next, const void* ctx),
                             const void* ctx) {
    uint8_t* fixed = (uint8_t*)calloc((size_t)(l1 > l0 ? l1 - l0 : 1), 1);
#pragma omp parallel
    {
        float* z = (float*)malloc(sizeof(float) * (size_t)N);
        float* o = (float*)malloc(sizeof(float) * (size_t)N);
#pragma omp for schedule(dynamic, 1)
        for (int32_t l = l0; l < l1; ++l) { /* layers are independent here */
            uint8_t f = 0;
            for (int32_t k = 0; k < N; ++k) z[k] = 0.0f;
            eval(l, z, o, ctx);
            if (row_all_equal(o, N, 0.0f)) f |= 1;
            for (int32_t k = 0; k < N; ++k) z[k] = ymax;
            eval(l, z, o, ctx);
            if (row_all_equal(o, N, ymax)) f |= 2;
            fixed[l - l0] = f;
        }
        free(z);
        free(o);
    }
    return fixed;
}

static int64_t layers_fast(int32_t N, float ymax, int32_t l0, int32_t l1, int64_t B, const float* Yin, float* Yout,
                           int32_t nthreads, void (*eval)(int32_t, const float*, float*, const void*),
                           const void* ctx) {
    set_threads(nthreads);
    uint8_t* fixed = fixed_points(N, l0, l1, ymax, eval, ctx);
    int64_t skipped = 0;
#pragma omp parallel reduction(+ : skipped)
    {
        float* a = (float*)malloc(sizeof(float) * (size_t)N);
        float* c = (float*)malloc(sizeof(float) * (size_t)N);
#pragma omp for schedule(dynamic, 4)
        for (int64_t r = 0; r < B; ++r) {
            memcpy(a, Yin + r * N, sizeof(float) * (size_t)N);
            int kind = -1; /* what `a` is: -1 not yet checked, 0 other, 1 all-zero, 2 all-YMAX */
            for (int32_t l = l0; l < l1; ++l) {
                const uint8_t f = fixed[l - l0];
                if (f && kind < 0)
                    kind = row_all_equal(a, N, 0.0f) ? 1 : (row_all_equal(a, N, ymax) ? 2 : 0);
                if (kind > 0 && (f & kind)) {
                    skipped += 1;  /* the layer maps this row to itself: `a` unchanged, `kind` still holds */
                    continue;
                }
                eval(l, a, c, ctx);
                float* tmp = a; a = c; c = tmp;
                kind = -1;
            }
            memcpy(Yout + r * N, a, sizeof(float) * (size_t)N);
        }
        free(a);
        free(c);
    }
    free(fixed);
    return skipped;
}

struct csc_ctx { int32_t N; const int64_t* ptr; const int32_t* idx; const float* val; const float* bias; float ymax; };
static void eval_csc(int32_t l, const float* y, float* y_next, const void* vctx) {
    const struct csc_ctx* x = (const struct csc_ctx*)vctx;
    row_layer_f32(x->N, x->ptr + (int64_t)l * (x->N + 1), x->idx, x->val, x->bias + (int64_t)l * x->N, x->ymax, y,
                  y_next);
}
struct circ_ctx { int32_t N, K; const int32_t* nu; const float* w; const float* bias; float ymax; };
static void eval_circ(int32_t l, const float* y, float* y_next, const void* vctx) {
    const struct circ_ctx* x = (const struct circ_ctx*)vctx;
    row_layer_circ_f32(x->N, x->K, x->nu[l], x->w + (int64_t)l * x->K, x->bias + (int64_t)l * x->N, x->ymax, y,
                       y_next);
}

int64_t oracle_layers_f32_fast(int32_t N, const int64_t* ptr, const int32_t* idx, const float* val,
                               const float* bias, float ymax, int32_t l0, int32_t l1,
                               int64_t B, const float* Yin, float* Yout, int32_t nthreads) {
    struct csc_ctx x = {N, ptr, idx, val, bias, ymax};
    return layers_fast(N, ymax, l0, l1, B, Yin, Yout, nthreads, eval_csc, &x);
}

int64_t oracle_layers_circulant_f32_fast(int32_t N, int32_t K, const int32_t* nu, const float* w,
                                         const float* bias, float ymax, int32_t l0, int32_t l1, int64_t B,
                                         const float* Yin, float* Yout, int32_t nthreads) {
    struct circ_ctx x = {N, K, nu, w, bias, ymax};
    return layers_fast(N, ymax, l0, l1, B, Yin, Yout, nthreads, eval_circ, &x);
}

/* Sum downsampling: "divides the original column into n segments, each containing N/n elements
 * ... For each segment, we run a simple sum reduction". */
void oracle_sum_downsample(int32_t N, int32_t n, int32_t s, const float* rows, double* F) {
    if (n <= 0) n = N;
    int32_t seg = N / n;
    for (int32_t q = 0; q < s; ++q) {
        for (int32_t g = 0; g < n; ++g) {
            int32_t k0 = g * seg, k1 = (g == n - 1) ? N : (g + 1) * seg;
            double sum = 0.0;
            for (int32_t k = k0; k < k1; ++k) sum += (double)rows[(int64_t)q * N + k];
            F[(int64_t)g * s + q] = sum;
        }
    }
}

/* Alg. 1, serialised: the parallel threads of lines 13-14 each evaluate one
 * (segment, column) pair of Eq. (2); the atomicAdd of line 14 is the count below. */
int32_t oracle_prune(int32_t n, int32_t s, const double* F, float eta, float eps, int32_t* col_idx) {
    int32_t* tmp_idx = (int32_t*)malloc(sizeof(int32_t) * (size_t)s); /* line 2 */
    double* base = (double*)malloc(sizeof(double) * (size_t)n);
    for (int32_t q = 0; q < s; ++q) tmp_idx[q] = col_idx[q];        /* lines 3-4 */
    const double thr = (double)n * (double)eps;
    for (int32_t cmp = 0; cmp < s; ++cmp) {                           /* line 6 */
        if (tmp_idx[cmp] == -1) continue;                             /* line 7 */
        for (int32_t g = 0; g < n; ++g) base[g] = F[(int64_t)g * s + tmp_idx[cmp]]; /* lines 8-9 */
        for (int32_t q = 0; q < s; ++q) {
            if (q == cmp || tmp_idx[q] == -1) continue;               /* lines 13, 16 */
            int32_t diff = 0;                                         /* lines 10-11 */
            for (int32_t g = 0; g < n; ++g)                           /* Eq. (2), reading R2 */
                if (fabs(F[(int64_t)g * s + q] - base[g]) > (double)eta) diff += 1;
            if ((double)diff < thr) tmp_idx[q] = -1;                  /* lines 16-17 */
        }
    }
    int32_t cnt = 0;
    for (int32_t q = 0; q < s; ++q) {                                 /* lines 19-20 */
        col_idx[q] = tmp_idx[q];
        if (tmp_idx[q] != -1) ++cnt;
    }
    free(tmp_idx);
    free(base);
    return cnt;
}

/* Eq. (3)-(4), Alg. 2: L0 distance = number of elements that differ (Alg. 2 lines 10-12). */
void oracle_map_residual(int32_t N, int64_t R, const float* Y, const uint8_t* live, int32_t C,
                         const int32_t* cent, int32_t* M, float* Yhat, uint8_t* ne) {
    for (int64_t r = 0; r < R; ++r) {
        const float* y = Y + r * N;
        if (live && !live[r]) { M[r] = -2; ne[r] = 0; continue; }
        int is_cent = 0;
        for (int32_t c = 0; c < C; ++c) if (cent[c] == r) is_cent = 1;
        if (is_cent) {                                  /* Eq. (4) second case; M = -1 */
            M[r] = -1;
            memcpy(Yhat + r * N, y, sizeof(float) * (size_t)N);
            ne[r] = 1;                                  /* R7 */
            continue;
        }
        int64_t dist = (int64_t)N + 1;                  /* Alg. 2 line 3 */
        int32_t cluster = -1;
        for (int32_t c = 0; c < C; ++c) {               /* line 4 */
            const float* yc = Y + (int64_t)cent[c] * N;
            int64_t this_dist = 0;                      /* line 5 */
            for (int32_t k = 0; k < N; ++k)
                if (yc[k] != y[k]) this_dist += 1;      /* lines 11-12 */
            if (this_dist < dist) { dist = this_dist; cluster = c; } /* lines 14-16 */
        }
        if (cluster < 0) { M[r] = -2; ne[r] = 0; continue; } /* no centroid at all (C == 0) */
        const float* yc = Y + (int64_t)cent[cluster] * N;
        for (int32_t k = 0; k < N; ++k) Yhat[r * N + k] = y[k] - yc[k]; /* lines 17-20 */
        M[r] = cent[cluster];                           /* line 25 */
        ne[r] = (dist == 0) ? 0 : 1;                    /* lines 26-29 */
    }
}

/* one fp32 fma chain for output j over the stored order (same rule as Eq. (1) above) */
static float spmv_col_f32(const int64_t* p, const int32_t* idx, const float* val, const float* y, int32_t j) {
    float acc = 0.0f;
    for (int64_t e = p[j]; e < p[j + 1]; ++e) acc = fmaf(y[idx[e]], val[e], acc);
    return acc;
}

void oracle_post_layer(int32_t N, const int64_t* ptr, const int32_t* idx, const float* val,
                       const float* bias, float ymax, int32_t l, int64_t R, const int32_t* M,
                       const float* Yhat_in, uint8_t* ne, float* Yhat_out, float prune_eps,
                       int32_t nthreads) {
    const int64_t* p = ptr + (int64_t)l * (N + 1);
    const float* b = bias + (int64_t)l * N;
    set_threads(nthreads);
#pragma omp parallel for schedule(dynamic, 4)
    for (int64_t r = 0; r < R; ++r) {
        if (M[r] == -2) continue;
        if (M[r] == -1) {                               /* Eq. (5) first case; Alg. 3 lines 2-6 */
            for (int32_t j = 0; j < N; ++j) {
                float a_c = spmv_col_f32(p, idx, val, Yhat_in + r * N, j);
                Yhat_out[r * N + j] = sigma_f32(a_c + b[j], ymax);
            }
            ne[r] = 1;
            continue;
        }
        if (!ne[r]) continue;                           /* not in ne_idx */
        const float* yc = Yhat_in + (int64_t)M[r] * N;  /* centroid's Yhat(i) */
        int64_t count = 0;                              /* Alg. 3 line 7 */
        for (int32_t j = 0; j < N; ++j) {               /* Eq. (5) second case; Alg. 3 lines 8-11 */
            float a_c = spmv_col_f32(p, idx, val, yc, j);
            float a_r = spmv_col_f32(p, idx, val, Yhat_in + r * N, j);
            float v = sigma_f32((a_c + a_r) + b[j], ymax) - sigma_f32(a_c + b[j], ymax);
            if (prune_eps > 0.0f && fabsf(v) <= prune_eps) v = 0.0f;
            Yhat_out[r * N + j] = v;
            if (v != 0.0f) count += 1;
        }
        ne[r] = (count != 0) ? 1 : 0;                   /* lines 12-13 */
    }
}

/* Eq. (6): "We simply reverse Equation (4)". */
void oracle_recover(int32_t N, int64_t R, const int32_t* M, const uint8_t* ne, const float* Yhat,
                    float* Y_out, uint8_t* cat) {
    for (int64_t r = 0; r < R; ++r) {
        float* y = Y_out + r * N;
        for (int32_t j = 0; j < N; ++j) {
            float v;
            if (M[r] == -1) v = Yhat[r * N + j];
            else if (M[r] == -2) v = 0.0f;
            else v = (ne[r] ? Yhat[r * N + j] : 0.0f) + Yhat[(int64_t)M[r] * N + j];
            y[j] = v;
        }
        if (cat) {
            int any = 0;
            for (int32_t j = 0; j < N; ++j) if (y[j] != 0.0f) any = 1;
            cat[r] = (uint8_t)any;
        }
    }
}

static int row_is_zero(const float* y, int32_t N) {
    for (int32_t k = 0; k < N; ++k) if (y[k] != 0.0f) return 0;
    return 1;
}

int32_t oracle_snicit(int32_t N, int32_t L, const int64_t* ptr, const int32_t* idx,
                      const float* val, const float* bias, float ymax, int64_t B, const float* Y0,
                      int32_t t, int32_t s, int32_t n_seg, float eta, float eps, float prune_eps,
                      int32_t drop_dead, float* Y_out, uint8_t* cat, int32_t* M_out, int32_t* cent_out,
                      int32_t* n_cent_out, double* F_out, uint8_t* live_t, uint8_t* ne_final,
                      int32_t nthreads) {
    if (N <= 0 || L < 0 || B < 0 || t < 0 || s < 1) return -1;
    if (t > L) t = L;
    /* dead_ok[l]: every bias of layers l..L-1 is <= 0, so a zero row stays zero (R23) */
    uint8_t* dead_ok = (uint8_t*)malloc((size_t)L + 1);
    dead_ok[L] = 1;
    for (int32_t l = L - 1; l >= 0; --l) {
        int ok = dead_ok[l + 1];
        for (int32_t j = 0; j < N; ++j) if (bias[(int64_t)l * N + j] > 0.0f) ok = 0;
        dead_ok[l] = (uint8_t)ok;
    }
    size_t bytes = sizeof(float) * (size_t)B * (size_t)N;
    float* Y = (float*)malloc(bytes ? bytes : 1);
    float* Z = (float*)malloc(bytes ? bytes : 1);
    uint8_t* live = (uint8_t*)malloc((size_t)B + 1);
    memcpy(Y, Y0, bytes);
    for (int64_t r = 0; r < B; ++r)
        live[r] = (drop_dead && dead_ok[0] && row_is_zero(Y + r * N, N)) ? 0 : 1;

    /* Pre-convergence, Eq. (1) for i = 0..t-1 */
    for (int32_t l = 0; l < t; ++l) {
        oracle_layers_f32(N, ptr, idx, val, bias, ymax, l, l + 1, B, Y, Z, nthreads);
        float* tmp = Y; Y = Z; Z = tmp;
        if (drop_dead && dead_ok[l + 1])
            for (int64_t r = 0; r < B; ++r)
                if (live[r] && row_is_zero(Y + r * N, N)) live[r] = 0;
    }
    if (live_t) memcpy(live_t, live, (size_t)B);

    int32_t* M = (int32_t*)malloc(sizeof(int32_t) * (size_t)(B + 1));
    uint8_t* ne = (uint8_t*)malloc((size_t)B + 1);
    if (t >= L) {                                       /* no conversion: the plain path */
        for (int64_t r = 0; r < B; ++r) { M[r] = live[r] ? -1 : -2; ne[r] = live[r]; }
        if (n_cent_out) *n_cent_out = 0;
    } else {
        /* Column sampling: "simply take the first s columns", R14 */
        int32_t ss = 0;
        int32_t* sample = (int32_t*)malloc(sizeof(int32_t) * (size_t)s);
        for (int64_t r = 0; r < B && ss < s; ++r) if (live[r]) sample[ss++] = (int32_t)r;
        int32_t n = (n_seg <= 0) ? N : n_seg;
        float* rows = (float*)malloc(sizeof(float) * (size_t)(ss ? ss : 1) * (size_t)N);
        for (int32_t q = 0; q < ss; ++q) memcpy(rows + (int64_t)q * N, Y + (int64_t)sample[q] * N, sizeof(float) * (size_t)N);
        double* F = (double*)malloc(sizeof(double) * (size_t)n * (size_t)(ss ? ss : 1));
        oracle_sum_downsample(N, n, ss, rows, F);
        if (F_out) memcpy(F_out, F, sizeof(double) * (size_t)n * (size_t)ss);
        int32_t* col_idx = (int32_t*)malloc(sizeof(int32_t) * (size_t)(ss ? ss : 1));
        for (int32_t q = 0; q < ss; ++q) col_idx[q] = q;
        oracle_prune(n, ss, F, eta, eps, col_idx);
        /* "discard all the -1s from col_idx and sort the remaining" */
        int32_t C = 0;
        int32_t* cent = (int32_t*)malloc(sizeof(int32_t) * (size_t)(ss ? ss : 1));
        for (int32_t q = 0; q < ss; ++q) if (col_idx[q] != -1) cent[C++] = sample[col_idx[q]];
        for (int32_t a = 1; a < C; ++a)                 /* insertion sort (already ascending) */
            for (int32_t b2 = a; b2 > 0 && cent[b2 - 1] > cent[b2]; --b2) {
                int32_t x = cent[b2]; cent[b2] = cent[b2 - 1]; cent[b2 - 1] = x;
            }
        if (cent_out) memcpy(cent_out, cent, sizeof(int32_t) * (size_t)C);
        if (n_cent_out) *n_cent_out = C;
        oracle_map_residual(N, B, Y, live, C, cent, M, Z, ne);
        { float* tmp = Y; Y = Z; Z = tmp; }            /* Y now holds Yhat(t) */
        /* Post-convergence, Eq. (5) for i = t..l-1 */
        for (int32_t l = t; l < L; ++l) {
            oracle_post_layer(N, ptr, idx, val, bias, ymax, l, B, M, Y, ne, Z, prune_eps, nthreads);
            float* tmp = Y; Y = Z; Z = tmp;
        }
        free(sample); free(rows); free(F); free(col_idx); free(cent);
    }
    /* Final results recovery, Eq. (6) */
    float* out = Y_out ? Y_out : Z;
    if (t >= L) {
        for (int64_t r = 0; r < B; ++r)
            for (int32_t j = 0; j < N; ++j) out[r * N + j] = live[r] ? Y[r * N + j] : 0.0f;
        if (cat)
            for (int64_t r = 0; r < B; ++r) cat[r] = (uint8_t)!row_is_zero(out + r * N, N);
    } else {
        oracle_recover(N, B, M, ne, Y, out, cat);
    }
    if (M_out) memcpy(M_out, M, sizeof(int32_t) * (size_t)B);
    if (ne_final) memcpy(ne_final, ne, (size_t)B);
    free(Y); free(Z); free(live); free(M); free(ne); free(dead_ok);
    return 0;
}
