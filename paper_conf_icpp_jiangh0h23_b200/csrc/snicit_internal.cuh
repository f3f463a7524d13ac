// snicit_internal.cuh -- internal declarations of libsnicit.so (sm_100a).
// Kernel/launcher interfaces shared by the .cu files of the library; not part of the ABI.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

namespace snicit {

// ------------------------------------------------------------------ PTX helpers (TMA bulk, mbarrier)
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
// try_wait suspends the thread in hardware until the phase completes or the hint (ns) expires,
// so waiting warps do not burn issue slots spinning.
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity), "r"(1000000u)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    while (!mbar_try_wait(bar, parity)) {
    }
}
// 1-D bulk copy global -> shared (TMA engine, UBLKCP), completion counted on `bar`.
__device__ __forceinline__ void bulk_g2s(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(sdst)),
        "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}
// 1-D bulk copy shared -> global (TMA store), bulk-group completion.
__device__ __forceinline__ void bulk_s2g(void* gdst, const void* ssrc, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gdst), "r"(smem_u32(ssrc)),
                 "r"(bytes)
                 : "memory");
}
// acquire load of a flag written by another agent (copy engine / other kernel), gpu scope
__device__ __forceinline__ int ld_acquire_gpu(const int* p) {
    int v;
    asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
// order generic-proxy observations before later async-proxy (TMA) global accesses
__device__ __forceinline__ void fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
// L2 prefetch of a global range (TMA engine, no completion tracking)
__device__ __forceinline__ void bulk_prefetch_l2(const void* gsrc, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(gsrc), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read1() { asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// packed fp32x2 (sm_100+): each lane of the pair is an ordinary round-to-nearest fma/add, so a chain
// evaluated with fma2 is bit-identical to the same chain with fmaf (FFMA2 / FADD2 in SASS).
__device__ __forceinline__ unsigned long long f2_pack(float lo, float hi) {
    unsigned long long r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
    return r;
}
__device__ __forceinline__ void f2_unpack(unsigned long long r, float& lo, float& hi) {
    asm("mov.b64 {%0, %1}, %2;" : "=f"(lo), "=f"(hi) : "l"(r));
}
__device__ __forceinline__ unsigned long long f2_fma(unsigned long long a, unsigned long long b,
                                                     unsigned long long c) {
    unsigned long long d;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
    return d;
}
__device__ __forceinline__ unsigned long long f2_add(unsigned long long a, unsigned long long b) {
    unsigned long long d;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
}

// sigma(x) = min(max(x, 0), ymax): Table 2
__device__ __forceinline__ float sigma(float x, float ymax) { return fminf(fmaxf(x, 0.0f), ymax); }

// ------------------------------------------------------------------ layer kernels
enum LayerMode : int {
    MODE_PLAIN = 0,     // Eq. 1: y' = sigma(acc + b)
    MODE_CENTROID = 1,  // Eq. 5 first case, also stores a_c = acc (pre-activation, no bias)
    MODE_RESIDUAL = 2   // Eq. 5 second case: sigma((a_c + acc) + b) - sigma(a_c + b)
};

struct LayerArgs {
    int N;
    const float* yin;       // rows of N fp32 (indexed by row id)
    float* yout;
    const int* rows;        // active row ids (list)
    const int* count;       // device: number of active rows
    const float* bias;      // [N] of this layer
    float ymax;
    uint8_t* flag_pos;      // nullable: any-non-zero of the row, indexed by list position
    uint8_t* flag_row;      // nullable: same, indexed by row id
    int* app_list;          // nullable: rows with a non-zero output are appended here (unordered)
    int* app_count;         //   ... at atomicAdd(app_count, n) (zero on entry)
    int* zero_count;        // nullable: set to 0 by the kernel (rotating append counters)
    int* row_ctr;           // column-streaming kernel with app_list: per list position, zero on entry
                            //   and on exit (warps of a row count in; the last one appends the row)
    float* a_out;           // CENTROID: a_c [row][N]
    const float* a_c;       // RESIDUAL: a_c [slot][N]
    const int* cslot;       // RESIDUAL: centroid slot of each row id
    float prune_eps;        // RESIDUAL: |v| <= prune_eps -> 0
    // ELL weights (n-major: entry n of column j at n*N + j)
    int K;                  // max entries per column
    const uint16_t* idx16;  // used when N <= 65536
    const int32_t* idx32;
    const float* val;       // nullable when uniform
    const uint8_t* len;     // nullable: per-column length (ragged); NULL = all K
    float w0;               // uniform value
    int uniform_bias;       // 1: bias[j] == bias[0] for all j of this layer
    // circulant: column j reads (j + n*nu) mod N, n = 0..K-1, weight w[n] (or w0)
    int nu;
    const float* wtab;      // K per-n weights (device), nullable when uniform
    const float* wtab_host; // the same K weights in host memory (kernels taking them as parameters)
    // constant-row mode of the pre-convergence per-layer path (R26; column and segmented kernels)
    unsigned* cmin;         // nullable: per list position, min / max output bits (init 0xffffffff / 0,
    unsigned* cmax;         //   restored by the consumer)
    int* clist;             // rows that became constant: row id, value, layer (append at *ccount)
    float* cval;
    int* clayer;
    int* ccount;
    int layer;              // index of this layer
    int dead_drop;          // an all-zero row after this layer is dead (drop && dead_ok[l + 1])
    // range prediction (R30) in constant-row mode: a row whose output range after this layer has
    // min >= thr_hi is the constant row YMAX at t, max <= thr_lo the zero row at t (dead when thr_dead);
    // it leaves with layer index thr_layer = t - 1.  thr_hi = +inf, thr_lo = -1: off
    float thr_hi, thr_lo;
    int thr_layer, thr_dead;
    // general-CSC row-interleaved kernel (kernels_gen.cu): load-time schedule of this layer, or goff NULL
    const uint16_t* gidx;   // per-tap input ids (N * gkp, padded taps -> the zero slot N)
    const float* gval;      // per-tap weights in the same layout (NULL: uniform w0)
    const uint16_t* gsched; // G = 16: output id of each quad slot
    int grl;                // outputs per warp instruction G (2, 4, 16)
    int gkp;                // taps per column, padded to a multiple of 4 (arrays hold ceil(gkp / 8) blocks)
};

struct LayerPlan {
    int kind;       // 0 = ELL, 1 = CIRC (whole rows staged), 2 = CIRC segmented (large rows)
    int K;
    int nu;         // CIRC
    bool uniform;   // all values equal (w0)
    bool ragged;    // column lengths differ
    bool ubias;     // bias[j] identical for all j (SDGC: a constant per benchmark, Table 1)
    bool col;       // CIRC, strided: PLAIN layers may use the column-streaming kernel
    float w0;
    size_t ell_off; // element offset of this layer in the ELL arrays
    size_t w_off;   // offset in the per-n weight table
    bool gen;       // has a schedule for the general-CSC row-interleaved kernel (kernels_gen.cu)
    int gkp;        // its taps per column (K padded to a multiple of 4)
    size_t gen_off; // entry offset of this layer in the schedule arrays (N * gkp entries)
    int gsched_idx; // RL = 8: index of this layer's N-entry block of quad slots
};

// Epilogue of one output q of one row (acc = the fma chain, b = bias[q]).  `valid` == false marks a
// discarded tail output (computed unguarded for speed, q clamped): it must not store anything.
template <int MODE>
__device__ __forceinline__ float epilogue(const LayerArgs& a, float acc, float b, int q, int row, int slot,
                                          bool valid = true) {
    if constexpr (MODE == MODE_RESIDUAL) {
        const float ac = __ldg(a.a_c + (size_t)slot * a.N + q);
        float v = sigma((ac + acc) + b, a.ymax) - sigma(ac + b, a.ymax);
        if (a.prune_eps > 0.0f && fabsf(v) <= a.prune_eps) v = 0.0f;
        return v;
    } else {
        if constexpr (MODE == MODE_CENTROID) {
            if (valid) a.a_out[(size_t)row * a.N + q] = acc;
        }
        return sigma(acc + b, a.ymax);
    }
}

// cached blocks-per-SM (sets the dynamic shared-memory attribute on first use)
cudaError_t blocks_per_sm(const void* kern, int threads, size_t smem, int* out);

// launchers (kernels_circ.cu / kernels_layer.cu); return cudaError_t of the launch
cudaError_t launch_layer_ell(const LayerArgs& a, int mode, int max_rows, int num_sms, cudaStream_t st);
// general-CSC row-interleaved kernel (kernels_gen.cu)
int gen_rows_per_tile(int N);
bool gen_enabled();  // SNICIT_GEN != "0" (A/B switch)
double gen_build_layer(int N, int G, int Kp, const std::vector<std::vector<int32_t>>& cidx,
                       const std::vector<std::vector<float>>& cval, uint16_t* idx, float* w, uint16_t* sched);
cudaError_t launch_layer_gen(const LayerArgs& a, int mode, int max_rows, int num_sms, cudaStream_t st);
cudaError_t launch_layer_circ(const LayerArgs& a, int mode, int max_rows, int num_sms, cudaStream_t st);
bool circ_supported(int N, int K, int nu);
// segmented circulant kernel (rows too large for kernels_circ.cu), kernels_circ_seg.cu
cudaError_t launch_layer_circ_seg(const LayerArgs& a, int mode, int max_rows, int num_sms, cudaStream_t st);
bool circ_seg_supported(int N, int K, int nu);
// column-streaming circulant kernel for strided layers (PLAIN mode), kernels_circ_col.cu
cudaError_t launch_layer_circ_col(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st);
bool circ_col_supported(int N, int K, int nu);
bool ell_smem_ok(int N);

// ------------------------------------------------------------------ fused post-convergence (kernels_post.cu)
// Per-layer descriptor, resident in device memory, read by the multi-layer kernels.
struct PostLayer {
    int kind;       // 0 = ELL, 1 = circulant
    int cls;        // circulant stride class (kernels_circ.cu)
    int nu, K;
    int uniform_w;  // 1: all weights == w0
    int ubias;      // 1: all biases == b0
    float w0, b0;
    const float* bias;  // [N]
    const float* wtab;  // [K] per-n weights (circulant, !uniform_w)
    const uint16_t* idx16;
    const int32_t* idx32;
    const float* val;   // ELL values (n-major) or NULL when uniform
    const uint8_t* len; // ragged column lengths or NULL
};

struct PostArgs {
    int N, L, t;
    float ymax, prune_eps;
    int force_ell;            // 1: evaluate every layer with the general (ELL) gather
    const PostLayer* layers;  // device array [L]
    // centroid trajectory: rows cbuf[0..C) hold Yhat_c(t) on entry and Yhat_c(L) on exit
    float* cbuf;
    const int* n_cent;
    float* a_all;  // [(L - t)][s][N] pre-activations a_c per post layer, or NULL
    int s;
    // residual rows: rlist[0..*rcount) rows of yhat (Yhat_r(t) on entry, Yhat_r(L) on exit if alive)
    const int* rlist;
    const int* rcount;
    int* work_counter;  // zero on entry
    float* yhat;
    const int* cslot;
    uint8_t* ne_row;     // set to the row's final ne (0 once its residue became empty)
    int* alive_count;    // += 1 per row still non-empty at L (may be NULL)
    const int* cdone;    // nullable: centroid c already carried to L by centroid_const_kernel (skip it)
    int* cfrom;          // nullable: per centroid, first post layer (l - t) with a constant a_c row
    int scalar_ok;       // every post layer circulant with uniform weight and bias: constant residue rows
                         //   over constant centroids are carried by a scalar (residual_traj_kernel)
    int res_sparse;      // 1: sparse-entry residue form for residue rows with few non-zeros (circulant layers)
    const int* rnnz;     // nullable: non-zeros of each row's residue at t (map_residual), by row id
    int smem_floats;     // set by the launcher: dynamic shared memory of the kernel (floats)
    float* acs;          // nullable: [s][L - t] constant a_c values of each centroid from cfrom on (acconst)
    const float2* wb;    // nullable: [L] (w0, b0) of each layer (uniform layers)
    unsigned long long* dyn;  // nullable: [L - t + 1] residue rows by post layers survived, [L - t + 1] by the
                              //   post layer from which they were carried by a scalar (L - t: never)
    unsigned long long* ctr64;  // nullable: work counters (Ctr64)
};
// 64-bit work counters of one infer (stats): residue entries at t, residue row-layers by form, outputs
// evaluated by the sparse-entry form
enum Ctr64 : int { C64_RES_NNZ = 0, C64_FULL_RL, C64_SPARSE_RL, C64_SPARSE_OUT, C64_SCALAR_RL, C64_MAP_ROWS, C64_N };
cudaError_t launch_acconst(const PostArgs& a, int C_max, cudaStream_t st);
int post_fused_max_n();
cudaError_t launch_centroid_traj(const PostArgs& a, int C_max, cudaStream_t st);
// cluster (DSMEM) centroid trajectory: cls[l] = circulant stride class of layer l or -1
bool centroid_cluster_ok(int N, const int* nu, const int* cls, int t, int L);
cudaError_t launch_centroid_cluster(const PostArgs& a, int C_max, int win_max, cudaStream_t st);
cudaError_t launch_residual_traj(const PostArgs& a, int max_rows, int num_sms, cudaStream_t st);
// dynamic t: S probe rows through layers 0..tmax-1 (one CTA each); out[l][b] = (hash, live) after layer l
cudaError_t launch_probe_traj(const PostArgs& a, const float* rows, int S, int tmax, unsigned long long* out,
                              cudaStream_t st);
// constant centroid rows through layers t..L-1 that are all circulant with uniform weights and bias:
// one scalar chain per layer (exact, see kernels_post.cu); cout[c] = row at L, a.a_all filled if set,
// cdone[c] = 1 and ++*ndone for constant rows, cdone[c] = 0 otherwise
cudaError_t launch_centroid_const(const PostArgs& a, float* cout, int* cdone, int* ndone, int C_max, cudaStream_t st);
int circ_class_of(int N, int nu);

// ------------------------------------------------------------------ row-resident pre-convergence (kernels_pre_fused.cu)
enum PfClass : int { PF_NU1 = 0, PF_STR = 1, PF_Q32 = 2 };
struct PreFusedLayer {
    int nu;
    int cls;        // PfClass
    float w0, b0;   // uniform weight / bias of the layer
    int dead_next;  // dead_ok[l + 1]: an all-zero row after this layer stays zero (R23)
    int ymax_fixed; // the constant row YMAX maps to YMAX (sigma(chain(YMAX) + b0) == YMAX, evaluated on
                    // the host with the kernel's fma order)
    int pad[2];
};
// range prediction (R30, exact): when layers 0..t-1 share one weight w0 >= 0 and one bias b0, every output
// is a monotone function of every input, so after k more layers each element of a row lies in
// [out^k(min), out^k(max)], out(m) = sigma(chain(m) + b0) the map of a constant row (host-evaluated with
// the kernels' fma order).  hi[k-1] = least m with out^k(m) == YMAX (+inf if none), lo[k-1] = greatest m
// with out^k(m) == 0 (-1 if none), k = 1..kRangeK (longer horizons use entry kRangeK: hi is
// non-increasing and lo non-decreasing in k, so the shorter horizon is the stricter test).  Returns
// false (tables off) when the layers differ or w0 < 0.
constexpr int kRangeK = 32;
bool range_tables(const PreFusedLayer* layers, int t, float ymax, float* hi, float* lo);
struct PreFusedArgs {
    int N, t, H;     // H: circular halo (floats) of every staged row, >= 64 and >= 31*nu of STR layers
    float ymax;
    int drop;        // drop dead rows (R23)
    int const_skip;  // carry constant rows by one scalar chain per layer (R26)
    int gen_str;     // some layer < t is STR with nu != 32 (runtime-stride body needed)
    int l2_prefetch; // two-buffer configurations: prefetch the next row into L2
    const float* yin;
    const uint32_t* ybits;  // non-null: input rows as packed bits (N/32 words per row, LSB first), value `one`
    float one;
    const int* ready;       // nullable: ready[c] != 0 once chunk c (rows [b (2^c - 1), b (2^(c+1) - 1)),
    int ready_rows;         //   b = ready_rows) is in ybits (uploaded by the copy engine while the kernel runs)
    float* yout;
    const int* rows;   // input list [*count]
    const int* count;
    int* app_list;     // rows alive at t, appended unordered (nullable)
    int* app_count;    //   zero on entry
    int* work;         // row scheduler, zero on entry
    float* ydead;                 // nullable: rows found dead (R23) get N zeros here (the caller's y_out)
    uint8_t* rconst;              // nullable: rconst[row] = 1, rval[row] = v for rows constant at t (R26)
    float* rval;
    unsigned long long* full_rl;  // nullable: [0] += full (non-constant) row-layer fma evaluations,
                                  //   [1] += rows whose layer 0 ran as a popcount table (R32)
    unsigned long long* dyn;      // nullable: [t + 1] rows by full-evaluation count, [t + 1] rows by end layer
    int range_pred;               // caller: allow the range prediction (R30)
    int win_bounds;               // caller: R34 window-sum bounds at stride-1 layers after a failed R31
    int popc0;                    // layer 0 of stride 1 as a popcount table (R32): 0 off, 1 every two-valued
                                  //   row, 2 packed rows only (the bitmap is given; measured faster only there)
    int thr_ok;                   // range prediction on (R30; set by launch_pre_fused: one weight >= 0 and
    int dead_t;                   //   one bias for every layer < t); dead_t = dead_ok[t]
    int* n_const;                 // nullable: += rows that became constant
};
// 0 if N is not supported (T = N/32 threads must be 32..512)
int pre_fused_threads(int N);
size_t pre_fused_smem(int N, int H);
bool pre_fused_str_halo(int N);  // STR layers need H >= 31*nu
constexpr int kPfMaxLayers = 2000;  // t limit of the row-resident kernel (descriptors in parameter space)
// layers: host descriptors of layers 0..t-1
cudaError_t launch_pre_fused(const PreFusedArgs& a, const PreFusedLayer* layers, int num_sms, cudaStream_t st);

// kernels_pre_pair.cu: the row-resident pre phase in the paired-half layout (the default form)
size_t pre_pair_smem(int N, int Hp);
int pre_pair_halo(int N, const PreFusedLayer* layers, int t);  // < 0: not supported
cudaError_t launch_pre_pair(const PreFusedArgs& a, const PreFusedLayer* layers, int num_sms, cudaStream_t st);

// kernels_pre_cluster.cu: the row-resident pre phase for large rows (N = 16384 / 32768 / 65536), a row
// split over a cluster of N / 8192 CTAs exchanging layer outputs through distributed shared memory
int pre_cluster_class(int N, int nu);  // < 0: layer stride not supported
bool pre_cluster_supported(int N);
size_t pre_cluster_smem(int N, int Hh);
cudaError_t launch_pre_cluster(const PreFusedArgs& a, const PreFusedLayer* layers, int num_sms, cudaStream_t st);

// kernels_const.cu: constant rows in the per-layer pre-convergence path (R26)
cudaError_t launch_const_split(const int* list_in, const int* count_in, unsigned* cmin, unsigned* cmax, int* list_out,
                               int* count_out, int* clist, float* cval, int* clayer, int* ccount, int layer,
                               int dead_drop, int max_rows, cudaStream_t st, const LayerArgs* thr = nullptr);
cudaError_t launch_const_finish(const int* clist, const float* cval, const int* clayer, const int* ccount,
                                const PreFusedLayer* layers, int t, float ymax, int drop, int N, float* y, int* live,
                                int* live_count, int num_sms, cudaStream_t st, uint8_t* rconst = nullptr,
                                float* rval = nullptr);

// kernels_convert.cu
cudaError_t launch_iota(int* out, int n, int* count_out, cudaStream_t st);
cudaError_t launch_fill_i32(int* out, int n, int v, cudaStream_t st);
cudaError_t launch_fill_u8(uint8_t* out, int n, uint8_t v, cudaStream_t st);
cudaError_t launch_row_nonzero(const float* y, int N, const int* rows, const int* count, uint8_t* flag_pos,
                               int max_rows, int num_sms, cudaStream_t st);
// clear != 0: flag_pos[0 .. *count_in) is zeroed after it is read; row_flags (nullable):
// row_flags[list_in[i]] = flag_pos[i] for every position i
cudaError_t launch_compact(const int* list_in, const int* count_in, const uint8_t* flag_pos, int* list_out,
                           int* count_out, int max_n, int* scratch, cudaStream_t st, int clear = 0,
                           uint8_t* row_flags = nullptr);
int compact_scratch_ints(int max_n);
cudaError_t launch_downsample(const float* y, int N, const int* rows, const int* count, int s, int n_seg,
                              double* F, cudaStream_t st);
cudaError_t launch_prune(const double* F, const int* count, int s, int n_seg, float eta, float eps,
                         const int* rows, int* cent, int* n_cent, int* s_eff, int* col_idx, int* D, cudaStream_t st);
cudaError_t launch_map_residual(const float* y, int N, const int* rows, const int* count, const int* cent,
                                const int* n_cent, int* M, int* cslot, uint8_t* ne_row, uint8_t* flag_pos,
                                float* yhat, float* cbuf, int max_rows, int num_sms, cudaStream_t st,
                                const uint8_t* rconst, const float* rval, unsigned long long* nnz_sum,
                                int* dist /* [max_rows][s] scratch */, int s, int* rnnz /* nullable, by row */,
                                int* need /* [max_rows] scratch */, int* need_count /* device int */);
cudaError_t launch_recover(int N, int R, int plain, const float* yfinal, const uint8_t* live_row, const int* M,
                           const int* cslot, const uint8_t* ne_row, const float* cbuf, float* y_out,
                           uint8_t* cat, int num_sms, cudaStream_t st, int dead_zeroed = 0,
                           const uint8_t* yt_rconst = nullptr, const float* rval = nullptr, const int* cdone = nullptr);
// packed binary rows -> fp32 rows: y[r][j] = bit j of row r ? one : 0 (snicit_infer_packed)
cudaError_t launch_unpack_bits(const uint32_t* bits, int R, int N, float one, float* y, int num_sms, cudaStream_t st);
cudaError_t launch_mark_rows(const int* rows, const int* count, uint8_t* flag_row, int max_rows, cudaStream_t st);
// dynamic t: convergence statistics of S probe rows (live, all identical, distinct by hash) -> out[3]
cudaError_t launch_probe_stat(const float* y, int S, int N, int* out, cudaStream_t st);
cudaError_t launch_export_categories(const int* catlist, const int* count, long long offset, long long* out,
                                     long long cap, cudaStream_t st);

}  // namespace snicit
