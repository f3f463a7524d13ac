/*
 * snicit.h -- C ABI of libsnicit.so: SNICIT sparse-DNN inference on NVIDIA B200 (sm_100a).
 *
 * SNICIT (Jiang, Huang, Yu, Ho; ICPP 2023).  Citations are PAPER.md line numbers
 * (P:<line>) of the paper text; readings R1..R23 are listed in DESIGN.md section 3.
 *
 * Problem (Eq. 1): Y(l+1) = sigma(Y(l) . W(l) + b(l)),
 * sigma(x) = min(max(x, 0), ymax) (Table 2).  SNICIT (Fig. 2) runs the
 * first t layers plainly, converts Y(t) into centroid rows + residue rows (Sec. 3.2,
 * P:445-815), propagates centroids and non-empty residues (Sec. 3.3, Eq. 5)
 * and recovers Y(L) (Eq. 6).  The category set (R13) is the ascending
 * list of rows of Y(L) with any non-zero.
 *
 * Layout (R1): activations are B x N row-major fp32, one row per sample (the paper's
 * column).  Layer l's weights are CSC over OUTPUT neurons: the inputs k of output j are
 * idx[ptr[l*(N+1)+j] .. ptr[l*(N+1)+j+1]) with values val[..], in ACCUMULATION order (R12:
 * acc = fmaf(y[k], w, acc) over the stored order, then + b[j], then clamp).
 *
 * Every compute step runs in hand-written CUDA kernels on the handle's device; there is no
 * CPU fallback: without a usable sm_100 device every call returns SNICIT_E_CUDA.
 *
 * Thread-safety: a handle is not thread-safe; distinct handles may be used concurrently.
 * Errors: every call returns snicit_status; snicit_last_error() gives a thread-local message.
 */
#ifndef SNICIT_H
#define SNICIT_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SNICIT_ABI_VERSION 6

typedef struct snicit_network snicit_network; /* opaque: owns device copies of W, b + workspace */

typedef enum {
    SNICIT_OK = 0,
    SNICIT_E_INVALID_ARG = -1, /* bad shape / pointer / parameter */
    SNICIT_E_BAD_SPARSE = -2,  /* index out of range, duplicate in a column, ptr not monotone */
    SNICIT_E_OOM = -3,         /* device allocation failed */
    SNICIT_E_CUDA = -4,        /* CUDA runtime error or no sm_100 device */
    SNICIT_E_STATE = -5,       /* e.g. categories requested before any infer */
    SNICIT_E_UNSUPPORTED = -6
} snicit_status;

typedef enum {
    SNICIT_CSC = 0, /* per output j: its inputs k (the paper's row j of W(i+1)) */
    SNICIT_CSR = 1  /* per input k: its outputs j; transposed on load, entries of each output
                       column then ordered by ascending k */
} snicit_format;

typedef enum {
    SNICIT_KERNEL_AUTO = 0, /* shift-invariant layers use the circulant kernel, others ELL */
    SNICIT_KERNEL_ELL = 1,  /* force the general gather kernel on every layer */
    SNICIT_KERNEL_CIRC = 2, /* require the circulant kernel (error if a layer is not eligible) */
    SNICIT_KERNEL_CIRC_SMEM = 3 /* as CIRC, but strided layers use the shared-memory staged kernels
                                   instead of the column-streaming kernel (A/B and parity tests) */
} snicit_kernel;

/* SNICIT parameters (s = 32, t = 30, n = 16, eps = eta = 0.03 for SDGC;
 * P:1460-1465 medium nets: no downsampling, s = 128). */
typedef struct {
    int32_t n_segments;     /* n of sum downsampling; 0 = none (n = N), R15 */
    float eta;              /* Eq. 2 threshold (absolute, R3) */
    float eps;              /* Alg. 1 line 16: prune if diff < n*eps */
    float prune_eps;        /* near-zero residual relaxation (R8); 0 = exact */
    int32_t drop_dead_rows; /* 1 = exact zero-row compaction (R23) */
    int32_t kernel;         /* snicit_kernel */
    int32_t timing;         /* 1 = record per-phase CUDA-event times for snicit_stats;
                               2 = also one event pair around every pre-convergence layer kernel
                               (snicit_layer_profile) */
    int32_t ne_interval;    /* per-layer post mode: host reads the active-residual count every this
                               many post layers (P:966-970 uses 200) and stops launching residual
                               work at 0; 0 = default (64) */
    int32_t post_mode;      /* 0 = fused: centroid rows and each residue row carried through all
                               post-convergence layers in shared memory (2 launches; rows leave when
                               their residue becomes empty); 1 = per layer: centroid layer + residue
                               layer + ne_idx row compaction for every layer.  Results are
                               identical.  N > 24576 always uses the per-layer mode. */
    int32_t post_cluster;   /* fused mode: 1 = each centroid row carried by a thread-block cluster of
                               8 CTAs exchanging layer outputs through distributed shared memory
                               (when every post layer is circulant and partition-compatible); 0 = one
                               CTA per centroid.  Results identical. */
    int32_t post_const;     /* 1 = a centroid row that is constant at t (all elements bitwise equal)
                               is carried through the post layers by one scalar fma chain per layer
                               when every post layer is circulant with uniform weights and bias
                               (such a layer maps a constant row to a constant row; bit-identical
                               results); 0 = always the full-row evaluation */
    int32_t pre_fused;      /* pre-convergence layers 0..t-1 (Eq. 1): 1 = row-resident fused kernel -- a
                               CTA keeps one row in shared memory for all t layers (Y0 read and Y(t)
                               written once) and carries a row that became constant (all elements
                               equal) by one scalar fma chain per layer (R26, exact); 2 = the same kernel
                               without the constant-row shortcut (every live row evaluated in full);
                               0 = one kernel launch per layer; 3 = as 1; 4 = the row-resident kernel with
                               each row split over a thread-block cluster of N/8192 CTAs exchanging layer
                               outputs through distributed shared memory (N = 16384 / 32768 / 65536; the
                               cluster form of a row that does not fit one CTA at several CTAs per SM);
                               5 = as 1 with the row stored as pairs (y[p], y[p + N/2]) read by 8-byte
                               loads (kernels_pre_pair.cu).  1 uses the cluster form of 4 for rows one CTA
                               cannot hold (N = 32768 / 65536); at N <= 16384, 4 and 5 are measured
                               alternatives (slower than 1 on B200), kept selectable
                               and parity-tested.
                               6 = as 1 with fma chains for every non-constant row-layer: without the
                               range prediction (R30/R31: a row whose output range or class-sum bounds
                               prove Y(t) the constant row YMAX or zero leaves early) and without the
                               popcount layer 0 (R32: a stride-1 layer 0 on a row of zeros and one value
                               is a table lookup by window count); 2 also runs without R32.  For
                               measurement.  R32 runs on packed rows (snicit_infer_packed: the bitmap is
                               given) and, with 1, on fp32 rows of zeros and one value when N = 2048..4096
                               (the bitmap built by ballots: faster there, slower at N = 1024 / 16384); 7 = as 1
                               with R32 on such fp32 rows at every N.  1 also uses
                               R34 (window-sum bounds of stride-1 layers) with R30 / R31.
                               Used when every layer < t is circulant
                               with 32 taps, uniform weight and uniform bias, and N/32 is one of
                               32..512 (N = 1024..16384) or N = 32768 / 65536 (cluster form, every
                               stride);
                               otherwise the per-layer kernels run.
                               Results are bit-identical in every mode (tested). */
    int32_t pre_const;      /* per-layer pre-convergence path (pre_fused = 0 or not applicable): 1 = a row
                               whose outputs are all equal leaves the active list and is carried by one
                               scalar fma chain per layer, written once at t (R26, exact; column-streaming
                               and segmented layer kernels, every layer < t circulant with uniform weight
                               and bias), and with every layer < t sharing one weight and bias a row
                               whose output range bounds Y(t) to YMAX or to zero leaves at once (R30,
                               exact); 2 = as 1 without R30; 0 = every live row through every layer */
    int32_t res_sparse;     /* fused post mode, circulant post layers: 1 = a residue row with few non-zero
                               entries propagates only them (the outputs they touch are evaluated, every
                               other output of Eq. 5 is exactly 0; north_star "only the nonzero residual
                               entries are propagated"), chosen per row and layer from its non-zero count;
                               0 = always the dense-row form.  Results identical. */
    int32_t dyn_t;          /* 1 = dynamic threshold layer (the paper's future work): the first s
                               rows of the batch are run through the layers on the side; with l* the first
                               layer after which all of them that are live are identical (one centroid, no
                               residue among them), t = min(2 l*, threshold_layer); if that never happens and
                               more than half of them are still distinct, the uncompressed path (t = L).
                               stats.threshold_layer reports the t used.  0 = t as given.  Results are the
                               plain result for any t (within the tolerance of SNICIT's Eq. 5 rounding). */
} snicit_options;

/* Per-run statistics of the last snicit_infer (times in ms, valid when options.timing). */
typedef struct {
    double t_pre_ms, t_convert_ms, t_post_ms, t_recover_ms, t_total_ms;
    int64_t batch;            /* rows of this call */
    int64_t live_at_t;        /* rows not dropped as dead at layer t */
    int64_t residual_at_t;    /* non-empty residue rows right after conversion */
    int64_t residual_final;   /* non-empty residue rows after the last layer */
    int64_t n_categories;
    int32_t n_centroids;      /* cent_cnt = |y*| */
    int32_t n_sampled;        /* s actually sampled (min(s, live)) */
    int32_t threshold_layer;  /* t used (min(t, L)) */
    int32_t circ_layers;      /* layers run by the circulant kernel */
    int64_t kernel_launches;  /* kernels launched by this infer */
    int32_t const_centroids;  /* centroids carried through the post layers as constant rows
                                 (options.post_const) */
    int32_t pre_fused;        /* the pre-convergence layers ran in the row-resident kernel: 1 = one CTA per
                                 row (kernels_pre_fused.cu), 2 = a cluster of CTAs per row
                                 (kernels_pre_cluster.cu), 0 = one launch per layer */
    int32_t pre_const_rows;   /* fused: rows that became constant before t (carried by a scalar) */
    int64_t pre_full_rows;    /* fused: full-row layer evaluations (row x layer, 32*N fma each) */
    int64_t res_nnz_at_t;     /* non-zero entries of the non-empty residue rows right after conversion */
    int64_t res_full_rl;      /* residue row-layers evaluated in the dense-row form (N outputs each) */
    int64_t res_sparse_rl;    /* residue row-layers evaluated in the sparse-entry form */
    int64_t res_sparse_out;   /* outputs evaluated by the sparse-entry form (32 fma each) */
    int64_t res_scalar_rl;    /* residue row-layers carried by a scalar (constant rows, R25/R26) */
    int64_t map_rows;         /* rows whose L0 distances to every centroid Alg. 2 computed (the others: centroid
                                 rows and constant rows with an equal constant centroid, R26) */
    double t_map_ms;          /* map_residual kernels (Alg. 2), CUDA events (options.timing), else -1 */
    double t_residual_ms;     /* residue trajectory kernel (Eq. 5, fused post mode), else -1 */
    int64_t pre_popc_rows;    /* fused: rows whose layer 0 (stride 1) ran as a popcount table lookup (a row
                                 of 0 and one value c: each output depends only on the count of c in its
                                 window, R32) -- not counted in pre_full_rows */
} snicit_stats_t;

/* Fill *opt with the paper's SDGC defaults (n = 16, eta = eps = 0.03, prune_eps = 0,
 * drop_dead_rows = 1, kernel = AUTO, timing = 0, ne_interval = 64, post_mode = 0, post_cluster = 1, post_const = 1,
 * pre_fused = 1, pre_const = 1). */
void snicit_default_options(snicit_options* opt);

/* Load a network (one-time; untimed in the benchmark).  All pointers are HOST pointers and
 * are copied (the caller may free them on return).  n_layers >= 1, n_neurons >= 1.
 * ptr: L*(N+1) int64 ABSOLUTE offsets into idx/val (layer l's first offset = layer l-1's last);
 * for SNICIT_CSR the roles of rows/columns swap (per input k).  bias: L*N fp32.  ymax > 0.
 * Validation: offsets monotone, 0 <= idx < N, no duplicate index within a column, finite
 * values -> SNICIT_E_BAD_SPARSE / SNICIT_E_INVALID_ARG.  cuda_device: device ordinal.
 * On success *out owns device memory until snicit_free_network. */
snicit_status snicit_load_network(int32_t n_neurons, int32_t n_layers, snicit_format fmt,
                                  const int64_t* ptr, const int32_t* idx, const float* val,
                                  const float* bias, float ymax, int32_t cuda_device,
                                  snicit_network** out);

/* Load a network given in the compact form of shift-invariant ("circulant") layers: column j of
 * layer l reads inputs (j + n*nu[l]) mod N, n = 0..K-1, in that order, with weight w[l*K + n] --
 * the RadiX-Net layers of SDGC, "sums of cyclic permutations".  Equivalent to
 * snicit_load_network with the explicit CSC (same plans, same results; tested) without the
 * L*N*K index arrays (C4: 32 GB).  Requirements: N % nu[l] == 0, K*nu[l] <= N (distinct inputs),
 * K == 32 (the circulant kernels' tap count) -> else SNICIT_E_BAD_SPARSE / SNICIT_E_UNSUPPORTED.
 * nu: L int32; w: L*K fp32; bias: L*N fp32 (host pointers, copied).  The general ELL kernel is
 * unavailable for such a handle (options.kernel = SNICIT_KERNEL_ELL -> SNICIT_E_UNSUPPORTED). */
snicit_status snicit_load_network_circulant(int32_t n_neurons, int32_t n_layers, const int32_t* nu,
                                            int32_t K, const float* w, const float* bias, float ymax,
                                            int32_t cuda_device, snicit_network** out);

/* All work of this handle is issued on `cuda_stream` (a cudaStream_t, e.g.
 * torch.cuda.current_stream().cuda_stream); NULL = the legacy default stream. */
snicit_status snicit_set_stream(snicit_network* net, void* cuda_stream);

/* Run inference on `batch` rows.
 *  y0:              batch*N fp32 row-major (R1); device pointer if y0_on_device else host.
 *                   Not modified.
 *  row_offset:      global id of local row 0 (multi-GPU row sharding); category
 *                   ids are row_offset + local row.
 *  threshold_layer: t; t >= L runs the uncompressed plain path.
 *  centroid_count:  s, the sample size and upper bound on cent_cnt; 1 <= s <= 1024
 *                   (larger: SNICIT_E_UNSUPPORTED).
 *  opt:             NULL = snicit_default_options.
 *  y_out:           batch*N fp32, caller-owned; device pointer if y_out_on_device else host;
 *                   NULL = do not materialise Y(L) (categories are still computed).  A device y_out
 *                   (not overlapping a device y0) also stores Y(t) when the row-resident pre phase runs,
 *                   so rows whose Y(L) equals their constant Y(t) are written once.
 * Alignment: device y0 / y_out must be 16-byte aligned (TMA bulk copies and float4 accesses);
 * otherwise SNICIT_E_INVALID_ARG.
 * Host synchronisation: when y0 or y_out is a HOST pointer the call returns only after the stream
 * has finished with it (y_out filled, y0 consumed).  With device pointers only, the work is queued
 * on the handle's stream and the call returns immediately (per-layer post mode may read a device
 * counter every opt->ne_interval layers).  snicit_categories synchronises the stream.
 * The caller's current CUDA device is restored on return (every entry point). */
snicit_status snicit_infer(snicit_network* net, const float* y0, int64_t batch,
                           int32_t y0_on_device, int64_t row_offset, int32_t threshold_layer,
                           int32_t centroid_count, const snicit_options* opt, float* y_out,
                           int32_t y_out_on_device);

/* snicit_infer for binary inputs given as a packed bitmap (the SDGC inputs are binary images,
 * P:297-302; 32x fewer bytes to upload than fp32 rows).  Row r of Y0 is
 *   Y0[r][j] = (y0_bits[r*W + j/32] >> (j % 32)) & 1 ? one_value : 0.0f,   W = ceil(N/32) words,
 * i.e. bit j%32 (LSB first) of 32-bit word j/32; bits of the last word beyond N are ignored.
 * y0_bits: batch*W uint32, device pointer if bits_on_device else host.  one_value: finite.
 * When the row-resident pre-convergence kernel applies (options.pre_fused, N % 128 == 0) it reads
 * each row's bits itself and expands them in shared memory (no fp32 Y0 in HBM); host bits are then
 * uploaded in geometrically growing chunks (512, 1024, 2048, ... rows) by the copy engine on a side
 * stream WHILE the kernel runs (it
 * waits per chunk on a ready flag), so the upload overlaps the compute (pinned host memory gives
 * the asynchronous copies; pageable memory works but the copies block the host).  Otherwise the
 * rows are copied, then unpacked by
 * a kernel into the handle's workspace.  Either way the inference proceeds exactly as snicit_infer
 * on the equivalent fp32 Y0 (same results, tested).  Host bits: the call returns once the upload has
 * consumed them (the buffer may then be reused).  Device bits must be 16-byte aligned.  All other
 * arguments as snicit_infer. */
snicit_status snicit_infer_packed(snicit_network* net, const uint32_t* y0_bits, int64_t batch,
                                  int32_t bits_on_device, float one_value, int64_t row_offset,
                                  int32_t threshold_layer, int32_t centroid_count,
                                  const snicit_options* opt, float* y_out, int32_t y_out_on_device);

/* Category ids of the last infer, ascending, as int64 global row ids (library-owned until
 * the next infer/free; copied out here).  Two-call pattern: rows == NULL -> *count = total.
 * Otherwise *count is the capacity of rows on entry and the number written on return
 * (min(capacity, total)).
 * rows_on_device != 0: rows is a device pointer (device-to-device copy, no host sync beyond
 * the count).  SNICIT_E_STATE before any infer. */
snicit_status snicit_categories(snicit_network* net, int64_t* rows, int64_t* count,
                                int32_t rows_on_device);

/* Device-side export of the category set of the last infer for the multi-GPU all-gather (SURVEY
 * 8(e)): asynchronous on the handle's stream, no host synchronisation.  out (DEVICE pointer, 8-byte
 * aligned, 1 + capacity int64): out[0] = total number of categories of this shard, out[1 + i] =
 * row_offset + local row id of the i-th category (ascending), i < min(total, capacity); the rest of
 * `out` is left untouched.  SNICIT_E_STATE before any infer. */
snicit_status snicit_categories_device(snicit_network* net, int64_t* out, int64_t capacity);

/* Statistics of the last infer (synchronises the stream). */
snicit_status snicit_stats(snicit_network* net, snicit_stats_t* out);

/* Per-launch profile of the pre-convergence layer kernels of the last infer run with
 * options.timing == 2: for layer i < *n (n = min(t, max)): ms[i] = CUDA-event duration of the
 * layer kernel launch (on the handle's stream), rows[i] = active rows it processed, bytes[i] =
 * algorithmic HBM bytes of the launch (8*rows*N + W bytes + 4*N; the
 * row-resident kernel: one launch, 4*N per input row + 4*N per row alive at t (+ 4*N per dead row
 * when it wrote the dead rows' zeros into a device y_out)).
 * Host pointers; any may be NULL.  Synchronises the stream. */
snicit_status snicit_layer_profile(snicit_network* net, int32_t max, double* ms, int64_t* rows, double* bytes,
                                   int32_t* n);

/* Per-layer dynamics of the last infer run with options.timing >= 1 (metrics / logging), for
 * layers l < *n = min(max, L) (host pointers, any may be NULL; -1 = not recorded for that layer):
 *  pre_full[l]   (l < t) rows evaluated in full by pre-convergence layer l (the others alive are carried as
 *                constant rows, R26);
 *  pre_live[l]   (l < t) rows alive after layer l: not dropped as dead (R23) -- the row-resident kernel drops a
 *                row at the layer by which it is proven zero, exactly (all outputs 0) or by the range rule
 *                (R30: its range bounds Y(t) to zero), so this counts rows not yet proven zero;
 *  res_alive[l]  (l >= t) non-empty residue rows after post-convergence layer l (ne_idx);
 *  res_scalar[l] (l >= t) residue rows carried by a scalar from post layer l or earlier.
 * Recorded by the row-resident pre phase and the fused post mode; the per-layer pre path reports pre_full
 * / pre_live from its per-layer active counts when options.timing == 2.  Synchronises the stream. */
snicit_status snicit_dynamics(snicit_network* net, int32_t max, int64_t* pre_full, int64_t* pre_live,
                              int64_t* res_alive, int64_t* res_scalar, int32_t* n);

/* ---- test hooks (used by tests/ for step-level parity; not needed by applications) ---- */

/* Clustering state of the last infer (t < L): centroid row ids (ascending, <= s entries),
 * cent_cnt, mapper M (batch int32: -1 centroid, -2 dead, else centroid row id), ne flags
 * at layer t (batch uint8), F (n x n_sampled fp64, row-major), live flags at t (batch uint8).
 * Any output pointer may be NULL.  Host pointers. */
snicit_status snicit_debug_clustering(snicit_network* net, int32_t* cent, int32_t* n_cent,
                                      int32_t* M, uint8_t* ne_t, double* F, int32_t* n_sampled,
                                      uint8_t* live_t);

/* One plain layer (Eq. 1) of the loaded network on `rows` device rows: yout = sigma(yin . W(l) + b(l)).
 * kernel: SNICIT_KERNEL_ELL, SNICIT_KERNEL_CIRC / SNICIT_KERNEL_CIRC_SMEM (error if not eligible) or AUTO.
 * yin, yout: device pointers, rows*N fp32, must not alias. */
snicit_status snicit_debug_layer(snicit_network* net, int32_t layer, const float* yin,
                                 float* yout, int64_t rows, int32_t kernel);

/* Range-prediction horizon tables (R30; host computation, no GPU needed): for a layer map of a
 * constant row out(v) = min(max(chain(v) + b0, 0), ymax), chain = 32 fmas acc = fma(v, w0, acc) from +0,
 * hi[k-1] = least v in [0, ymax] with out^k(v) == ymax (+inf if none) and lo[k-1] = greatest v with
 * out^k(v) == 0 (-1 if none), k = 1..kmax (kmax <= 32).  Returns 1 if either table is active, 0 if
 * neither (or w0 < 0), SNICIT_E_INVALID_ARG for bad arguments.  Host pointers, kmax floats each. */
int32_t snicit_debug_range_tables(float w0, float b0, float ymax, int32_t kmax, float* hi, float* lo);

/* Test hook (host only, no GPU needed): the load-time schedule of the general-CSC row-interleaved kernel
 * (kernels_gen.cu) for one layer of n_neurons outputs with K inputs each.
 * cols: n_neurons * K input indices, column-major per output (entry n of output j at j * K + n, chain
 * order).  Writes the number of outputs one warp instruction covers for this N (G = 2, 4 or
 * 16 -- tiles of 128 / G rows -- or 0 = kernel not used) to *rows_per_tile and the mean number of
 * shared-memory wavefronts per quarter-warp tap of the schedule to *cost (1.0 = conflict-free; G = 2 and
 * G = 4 read whole lines and are always 1.0).  Returns SNICIT_OK or SNICIT_E_INVALID_ARG. */
snicit_status snicit_debug_gen_schedule(int32_t n_neurons, int32_t K, const int32_t* cols, int32_t* rows_per_tile,
                                        double* cost);

/* 1 if layer l is eligible for the circulant kernel, 0 if not, < 0 on error. */
int32_t snicit_layer_is_circulant(const snicit_network* net, int32_t layer);

/* Release all device memory of the handle.  NULL is a no-op. */
void snicit_free_network(snicit_network* net);

/* Thread-local description of the last error ("" if none). */
const char* snicit_last_error(void);

/* SNICIT_ABI_VERSION of the loaded library. */
int32_t snicit_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SNICIT_H */
