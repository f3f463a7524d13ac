/*
 * oracle.h -- SNICIT CPU ORACLE.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may link or call this library.  It shares no code, header, table or helper with
 * the CUDA path (paper_conf_icpp_jiangh0h23_b200/csrc, include/snicit.h).
 *
 * Plain, slow, obviously-correct C.  Citations are PAPER.md line numbers
 * (/root/reference/PAPER.md; section / equation / algorithm named).  Readings of
 * ambiguous passages are numbered R1.. in DESIGN.md "Readings".
 *
 * Conventions (reading R1): activations are B x N row-major
 * (one row per sample = the paper's column of Y(i), Table 2).
 * A network has L layers; layer l (0-based, the paper's W(l+1)) is CSC over output
 * neurons: ptr[l*(N+1) + j] .. ptr[l*(N+1) + j + 1] are ABSOLUTE offsets into idx/val
 * listing the inputs k of output j, in accumulation order (reading R12).
 */
#ifndef SNICIT_ORACLE_H
#define SNICIT_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

int32_t oracle_version(void);

/* ---- Eq. (1), PAPER.md:435-438 (Sec. 3.1) and the SDGC problem statement PAPER.md:308-312:
 *      Y(l+1) = sigma(Y(l) . W(l) + b(l)),  sigma(x) = min(max(x, 0), ymax) (Table 2).
 * Layers [l0, l1) applied to B rows.  fp32: acc = +0; acc = fmaf(y[k], w, acc) over the stored
 * order; z = acc + b[j]; y'[j] = fminf(fmaxf(z, 0), ymax).  Rows are independent; OpenMP over
 * rows does not change any row's arithmetic.  nthreads <= 0: library default. */
void oracle_layers_f32(int32_t N, const int64_t* ptr, const int32_t* idx, const float* val,
                       const float* bias, float ymax, int32_t l0, int32_t l1,
                       int64_t B, const float* Yin, float* Yout, int32_t nthreads);

/* Same definition in fp64 (acc, bias add and clamp in double; input fp32 or previous fp64). */
void oracle_layers_f64(int32_t N, const int64_t* ptr, const int32_t* idx, const float* val,
                       const float* bias, float ymax, int32_t l0, int32_t l1,
                       int64_t B, const double* Yin, double* Yout, int32_t nthreads);

/* Eq. (1) for networks given in the compact circulant form (column j of layer l reads
 * (j + n*nu[l]) mod N, n = 0..K-1, weight w[l*K + n]): the same definition with the
 * index computed instead of stored; fp32, the same fma order as oracle_layers_f32 on the expanded
 * CSC (pinned against it in tests). */
void oracle_layers_circulant_f32(int32_t N, int32_t K, const int32_t* nu, const float* w, const float* bias,
                                 float ymax, int32_t l0, int32_t l1, int64_t B, const float* Yin, float* Yout,
                                 int32_t nthreads);

/* ---- Exact fast mode of Eq. (1) (used only to make full-size category parity
 * affordable).  A layer is a pure function of its input row, so a row equal (==) to a row whose
 * image was already computed has that image.  Two such rows are memoised per layer: the all-zero row
 * (its fma chains are +0 whatever the signs of its zeros) and the all-YMAX row.  When the image of
 * the all-zero (all-YMAX) row under layer l is that row again, every all-zero (all-YMAX) row is left
 * unchanged by layer l and the evaluation is skipped; every other row is evaluated exactly as by
 * oracle_layers_f32 / oracle_layers_circulant_f32 (same function calls).  Results are identical to
 * the plain mode (compared with ==; pinned in tests/test_oracle_pins.py).  Returns the number of
 * skipped row-layer evaluations. */
int64_t oracle_layers_f32_fast(int32_t N, const int64_t* ptr, const int32_t* idx, const float* val,
                               const float* bias, float ymax, int32_t l0, int32_t l1,
                               int64_t B, const float* Yin, float* Yout, int32_t nthreads);
int64_t oracle_layers_circulant_f32_fast(int32_t N, int32_t K, const int32_t* nu, const float* w,
                                         const float* bias, float ymax, int32_t l0, int32_t l1, int64_t B,
                                         const float* Yin, float* Yout, int32_t nthreads);

/* ---- Sum downsampling, Sec. 3.2.1, Fig. 3a PAPER.md:587-596.
 * rows: s x N (the sampled rows).  F: n x s row-major, F[g*s+q] = sum of rows[q][k] over
 * segment g, segments of floor(N/n) elements, last segment takes the remainder (R15).
 * Accumulated in fp64, ascending k (R3).  n == 0 means "no downsampling": n = N, F = rows^T. */
void oracle_sum_downsample(int32_t N, int32_t n, int32_t s, const float* rows, double* F);

/* ---- Sample pruning, Alg. 1 PAPER.md:687-716 with Eq. (2) PAPER.md:624-635 (reading R2):
 *   for cmp = 0..s-1 in order: if tmp_idx[cmp] != -1: base = F[:, cmp];
 *     for every q != cmp with tmp_idx[q] != -1:
 *        diff[q] = #{g : |F[g][q] - base[g]| > eta};  if diff[q] < n*eps: tmp_idx[q] = -1.
 * col_idx (length s) is input (0..s-1 on entry normally) and output (-1 = pruned).
 * eta, eps compared in fp64 ((double)eta, (double)n * (double)eps).  Returns #survivors. */
int32_t oracle_prune(int32_t n, int32_t s, const double* F, float eta, float eps, int32_t* col_idx);

/* ---- Mapper M and residue errors, Eq. (3), Eq. (4) PAPER.md:718-727,
 * Alg. 2 PAPER.md:777-815.  Y: R x N (layer-t activations), live[r] (0 = dead row dropped by
 * exact zero-row compaction, R23).  cent: C ascending centroid row ids.
 * Outputs: M[r] = -1 (centroid), -2 (dead), else argmin_c L0(Y_r - Y_c) with strict '<' over
 * cent in ascending order (first minimum wins, R6);  Yhat[r] = Y_r - Y_M(r) (fp32) for mapped
 * rows, Y_r for centroids, untouched for dead rows;  ne[r] = 1 for centroids, (dist != 0) for
 * mapped rows (R7), 0 for dead rows. */
void oracle_map_residual(int32_t N, int64_t R, const float* Y, const uint8_t* live, int32_t C,
                         const int32_t* cent, int32_t* M, float* Yhat, uint8_t* ne);

/* ---- Post-convergence update of one layer, Eq. (5), Alg. 3 PAPER.md:972-994.
 * Layer l of the network.  For centroid rows (M == -1): a_c[j] = fma-chain over the stored
 * order of Yhat_c; Yhat'_c = sigma(a_c + b).  For rows with M >= 0 and ne == 1:
 * a_r = fma-chain of Yhat_r;  Yhat'_r[j] = sigma((a_c[j] + a_r[j]) + b[j]) - sigma(a_c[j] + b[j])
 * with c = M[r] (Alg. 3 line 9 order, R12); ne'[r] = any_j Yhat'_r[j] != 0 (lines 10, 12-13).
 * Rows with ne == 0 (zero residual, absorbing: R16) or M == -2 are not touched.
 * prune_eps > 0: residual entries with |v| <= prune_eps set to 0 (near-zero relaxation,
 * PAPER.md:883-888, R8); 0 = exact. */
void oracle_post_layer(int32_t N, const int64_t* ptr, const int32_t* idx, const float* val,
                       const float* bias, float ymax, int32_t l, int64_t R, const int32_t* M,
                       const float* Yhat_in, uint8_t* ne, float* Yhat_out, float prune_eps,
                       int32_t nthreads);

/* ---- Final results recovery, Eq. (6), and categories (R13: a row is in the
 * category set iff its final row has any non-zero).  Y_out[r] = Yhat_r (centroid);
 * (ne ? Yhat_r : 0) + Yhat_M(r) (mapped);  0 (dead).  cat[r] = any_j Y_out[r][j] != 0. */
void oracle_recover(int32_t N, int64_t R, const int32_t* M, const uint8_t* ne, const float* Yhat,
                    float* Y_out, uint8_t* cat);

/* ---- The whole SNICIT pipeline (Fig. 2), composed from the steps above in
 * the paper's order; for small cases.  t >= L: no conversion (plain path).  drop_dead: exact
 * zero-row compaction (R23).  s: sample size (first s live rows, R14).  n_seg = n (0 = none).
 * Outputs (any may be NULL): Y_out (B x N), cat (B), M (B), cent (s) + n_cent, F (n x s),
 * live_t (B, live flags at layer t), ne_final (B).  Returns 0, or -1 on bad arguments. */
int32_t oracle_snicit(int32_t N, int32_t L, const int64_t* ptr, const int32_t* idx,
                      const float* val, const float* bias, float ymax, int64_t B, const float* Y0,
                      int32_t t, int32_t s, int32_t n_seg, float eta, float eps, float prune_eps,
                      int32_t drop_dead, float* Y_out, uint8_t* cat, int32_t* M, int32_t* cent,
                      int32_t* n_cent, double* F, uint8_t* live_t, uint8_t* ne_final,
                      int32_t nthreads);

#ifdef __cplusplus
}
#endif
#endif
