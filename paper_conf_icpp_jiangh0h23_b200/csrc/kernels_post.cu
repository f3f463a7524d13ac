// kernels_post.cu -- fused (multi-layer) post-convergence update, sm_100a.
//
// Eq. 5 (Alg. 3) for layers i = t..L-1 in two launches instead of ~3 per layer:
//
//  * centroid_traj_kernel: a centroid row evolves by Eq. 1 alone ("If a column in Yhat(i) is a
//    centroid, then we do not have to consider any errors"), independently of every
//    residue row.  One CTA per centroid keeps its row in shared memory for all L - t layers and
//    records the pre-activation a_c of every layer (needed by Eq. 5's second case).
//  * residual_traj_kernel: every residue row r is independent given a_c of its centroid M(r).  A CTA
//    takes a row from the non-empty list (ne_idx), keeps it in shared memory and applies
//    Yhat'_r = sigma((a_c + W.Yhat_r) + b) - sigma(a_c + b) layer after layer; the moment the row
//    becomes all-zero it leaves (ne_rec false, Alg. 3 lines 12-13).  A zero residue stays zero
//    (sigma((a_c + 0) + b) - sigma(a_c + b) == 0 exactly, reading R16), so this per-row early exit
//    returns exactly what per-layer ne_idx compaction returns.
//
// Per-layer arithmetic is identical to kernels_circ.cu / kernels_layer.cu (the stored-order fma
// chain, reading R12), so results are bit-identical to the per-layer path.
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include "snicit_internal.cuh"

namespace cg = cooperative_groups;

namespace snicit {

constexpr int kPostThreads = 256;
constexpr int kPK = 32;
constexpr int kPHalo = 64;  // circular halo of each staged row (nu == 1 windows, M + K - 1 = 48)

enum { PCLS_NU1 = 0, PCLS_Q32 = 1, PCLS_GEN = 2 };  // == CircClass of kernels_circ.cu

int post_fused_max_n() { return 24576; }  // 2 rows (+ halo) of shared memory per CTA

template <int MODE>
__device__ __forceinline__ float post_epi(float acc, float b, const float* ac, int q, float ymax, float prune_eps) {
    if constexpr (MODE == MODE_RESIDUAL) {
        const float c = __ldg(ac + q);
        float v = sigma((c + acc) + b, ymax) - sigma(c + b, ymax);
        if (prune_eps > 0.0f && fabsf(v) <= prune_eps) v = 0.0f;
        return v;
    } else {
        return sigma(acc + b, ymax);
    }
}

// The descriptor of one layer, held in registers (fields read once per layer).
struct PL {
    int kind, cls, nu, K, unif, ubias;
    float w0, b0;
    const float* bias;
    const float* wtab;
    const uint16_t* idx16;
    const int32_t* idx32;
    const float* val;
    const uint8_t* len;
};
__device__ __forceinline__ PL load_pl(const PostLayer* __restrict__ p) {
    PL r;
    r.kind = p->kind;
    r.cls = p->cls;
    r.nu = p->nu;
    r.K = p->K;
    r.unif = p->uniform_w;
    r.ubias = p->ubias;
    r.w0 = p->w0;
    r.b0 = p->b0;
    r.bias = p->bias;
    r.wtab = p->wtab;
    r.idx16 = p->idx16;
    r.idx32 = p->idx32;
    r.val = p->val;
    r.len = p->len;
    return r;
}

// One layer of one row by the whole CTA: in -> out (shared memory).  `dup` != 0: in[N .. 2N) holds a
// copy of in[0 .. N) (windows of every stride class read without wrap-around); else only a 64-float
// halo is present (nu == 1 windows) and the general class wraps explicitly.  Returns the number of
// this thread's outputs != 0; CENTROID mode also stores acc into aout (if non-NULL).
// MNU1 / MGEN: outputs per work item of the nu == 1 / general classes; QG: threads per residue class
// of the Q == 32 class (32 / QG outputs each).  Small values -> more, shorter items (latency-bound
// centroid trajectory on one SM); large -> fewer shared-memory loads per FMA (throughput).
template <int MODE, bool UNIF, int MNU1, int MGEN, int QG>
__device__ __forceinline__ int post_row_circ(const PL& Ld, int N, int dup, float ymax, float prune_eps,
                                              const float* __restrict__ in, float* __restrict__ out,
                                              const float* __restrict__ ac, float* __restrict__ aout, float& mn,
                                              float& mx) {
    const float w0 = Ld.w0, b0 = Ld.b0;
    const bool ubias = Ld.ubias != 0;
    const float* __restrict__ bias = Ld.bias;
    const int nu = Ld.nu, Q = N / nu;
    float w[UNIF ? 1 : kPK];
    if constexpr (!UNIF) {
#pragma unroll
        for (int n = 0; n < kPK; ++n) w[n] = __ldg(Ld.wtab + n);
    }
    int nz = 0;
    auto emit = [&](float acc, int q) {
        const float b = ubias ? b0 : __ldg(bias + q);
        if constexpr (MODE == MODE_CENTROID) {
            if (aout) aout[q] = acc;
        }
        const float v = post_epi<MODE>(acc, b, ac, q, ymax, prune_eps);
        out[q] = v;
        nz += (v != 0.0f);
        if constexpr (MODE == MODE_RESIDUAL) {
            mn = fminf(mn, v);
            mx = fmaxf(mx, v);
        }
    };
    if (Ld.cls == PCLS_NU1) {
        constexpr int M = MNU1, WIN = M + kPK - 1;
        const int items = (N + M - 1) / M;
        const bool exact = N % M == 0;
        for (int it = threadIdx.x; it < items; it += blockDim.x) {
            const int a0 = it * M;
            float R[WIN];
#pragma unroll
            for (int i = 0; i < WIN; ++i) R[i] = in[a0 + i];  // halo / copy: in[N + i] == in[i]
#pragma unroll
            for (int m = 0; m < M; ++m) {
                if (exact || a0 + m < N) {
                    float acc = 0.0f;
#pragma unroll
                    for (int n = 0; n < kPK; ++n) acc = fmaf(R[m + n], UNIF ? w0 : w[n], acc);
                    emit(acc, a0 + m);
                }
            }
        }
    } else if (Ld.cls == PCLS_Q32) {
        constexpr int OG = 32 / QG;  // outputs per item
        for (int it = threadIdx.x; it < nu * QG; it += blockDim.x) {
            const int c = it % nu;
            const int g0 = (it / nu) * OG;  // output group: a = g0 .. g0 + OG - 1
            const float* src = in + c;
            float R[32];  // rotated so that every index below is a compile-time constant
#pragma unroll
            for (int j = 0; j < 32; ++j) R[j] = src[((g0 + j) & 31) * nu];
#pragma unroll
            for (int mm = 0; mm < OG; ++mm) {
                float acc = 0.0f;
#pragma unroll
                for (int n = 0; n < kPK; ++n) acc = fmaf(R[(mm + n) & 31], UNIF ? w0 : w[n], acc);
                emit(acc, (g0 + mm) * nu + c);
            }
        }
    } else {
        constexpr int M = MGEN, WIN = M + kPK - 1;
        const int items = nu * ((Q + M - 1) / M);
        const bool exact = Q % M == 0;
        for (int it = threadIdx.x; it < items; it += blockDim.x) {
            const int c = it % nu;
            const int a0 = (it / nu) * M;
            const float* src = in + c;
            float R[WIN];
            if (dup || a0 + WIN <= Q) {
                const float* p = src + (size_t)a0 * nu;
#pragma unroll
                for (int i = 0; i < WIN; ++i) R[i] = p[i * nu];
            } else {
#pragma unroll
                for (int i = 0; i < WIN; ++i) {
                    int ai = a0 + i;  // < 3Q since Q >= K
                    ai = ai >= Q ? ai - Q : ai;
                    ai = ai >= Q ? ai - Q : ai;
                    R[i] = src[ai * nu];
                }
            }
#pragma unroll
            for (int m = 0; m < M; ++m) {
                if (exact || a0 + m < Q) {
                    float acc = 0.0f;
#pragma unroll
                    for (int n = 0; n < kPK; ++n) acc = fmaf(R[m + n], UNIF ? w0 : w[n], acc);
                    emit(acc, (a0 + m) * nu + c);
                }
            }
        }
    }
    return nz;
}

template <int MODE>
__device__ __forceinline__ int post_row_ell(const PL& Ld, int N, float ymax, float prune_eps,
                                             const float* __restrict__ in, float* __restrict__ out,
                                             const float* __restrict__ ac, float* __restrict__ aout, float& mn,
                                             float& mx) {
    const uint8_t* __restrict__ lens = Ld.len;
    const uint16_t* __restrict__ i16 = Ld.idx16;
    const int32_t* __restrict__ i32 = Ld.idx32;
    const float* __restrict__ val = Ld.val;
    const float* __restrict__ bias = Ld.bias;
    const int K = Ld.K;
    const bool unif = Ld.unif != 0, ubias = Ld.ubias != 0;
    const float w0 = Ld.w0, b0 = Ld.b0;
    int nz = 0;
    for (int j = threadIdx.x; j < N; j += blockDim.x) {
        const int len = lens ? (int)lens[j] : K;
        float acc = 0.0f;
        for (int n = 0; n < len; ++n) {
            const size_t e = (size_t)n * N + j;
            const int k = i16 ? (int)__ldg(i16 + e) : __ldg(i32 + e);
            const float w = unif ? w0 : __ldg(val + e);
            acc = fmaf(in[k], w, acc);
        }
        const float b = ubias ? b0 : __ldg(bias + j);
        if constexpr (MODE == MODE_CENTROID) {
            if (aout) aout[j] = acc;
        }
        const float v = post_epi<MODE>(acc, b, ac, j, ymax, prune_eps);
        out[j] = v;
        nz += (v != 0.0f);
        if constexpr (MODE == MODE_RESIDUAL) {
            mn = fminf(mn, v);
            mx = fmaxf(mx, v);
        }
    }
    return nz;
}

template <int MODE, int MNU1, int MGEN, int QG>
__device__ __forceinline__ int post_row_layer(const PL& Ld, int N, int dup, float ymax, float prune_eps,
                                               const float* in, float* out, const float* ac, float* aout,
                                               int force_ell, float& mn, float& mx) {
    if (Ld.kind == 1 && !force_ell) {
        if (Ld.unif)
            return post_row_circ<MODE, true, MNU1, MGEN, QG>(Ld, N, dup, ymax, prune_eps, in, out, ac, aout, mn, mx);
        return post_row_circ<MODE, false, MNU1, MGEN, QG>(Ld, N, dup, ymax, prune_eps, in, out, ac, aout, mn, mx);
    }
    return post_row_ell<MODE>(Ld, N, ymax, prune_eps, in, out, ac, aout, mn, mx);
}

__device__ __forceinline__ void stage_row(float* dst, const float* __restrict__ src, int N) {
    const float4* s4 = reinterpret_cast<const float4*>(src);
    float4* d4 = reinterpret_cast<float4*>(dst);
    for (int k = threadIdx.x; k < (N >> 2); k += blockDim.x) d4[k] = s4[k];
}
__device__ __forceinline__ void unstage_row(float* dst, const float* src, int N) {
    const float4* s4 = reinterpret_cast<const float4*>(src);
    float4* d4 = reinterpret_cast<float4*>(dst);
    for (int k = threadIdx.x; k < (N >> 2); k += blockDim.x) d4[k] = s4[k];
}
// row[N .. N + h) = row[0 .. h): h = N (full copy, `dup`) or the 64-float halo
__device__ __forceinline__ void fill_halo(float* row, int N, int h) {
    if ((h & 3) == 0 && (N & 3) == 0) {
        const float4* s4 = reinterpret_cast<const float4*>(row);
        float4* d4 = reinterpret_cast<float4*>(row + N);
        for (int i = threadIdx.x; i < (h >> 2); i += blockDim.x) d4[i] = s4[i];
    } else {
        for (int i = threadIdx.x; i < h; i += blockDim.x) row[N + i] = row[i];
    }
}
// staged row stride and halo: a full copy when two of them fit the shared-memory budget
__host__ __device__ inline int post_halo(int N) { return (size_t)N * 16 <= 200 * 1024 ? N : min(kPHalo, N); }

constexpr int kCentThreads = 1024;
// One CTA (1024 threads) per centroid row; items of 5 outputs (nu == 1: odd -> conflict-free LDS),
// 4 (general class) or 4 per residue
// class (Q == 32) so the whole SM works on every layer; the next layer's descriptor is loaded while
// the current layer computes (it is on the serial critical path otherwise).
__global__ void __launch_bounds__(kCentThreads) centroid_traj_kernel(PostArgs a) {
    extern __shared__ __align__(128) float sm[];
    const int C = *a.n_cent;
    const int c = blockIdx.x;
    if (c >= C || (a.cdone && a.cdone[c])) return;
    const bool want_a = a.a_all && (!a.rcount || *a.rcount > 0);  // a_c rows only for residue rows
    const int N = a.N;
    const int h = post_halo(N);
    const int dup = h == N;
    float* cur = sm;
    float* nxt = sm + N + h;
    stage_row(cur, a.cbuf + (size_t)c * N, N);
    __syncthreads();
    fill_halo(cur, N, h);
    __syncthreads();
    PL Ld = load_pl(a.layers + a.t);
    for (int l = a.t; l < a.L; ++l) {
        const PL Lnext = load_pl(a.layers + min(l + 1, a.L - 1));  // prefetch (serial critical path)
        float* aout = want_a ? a.a_all + ((size_t)(l - a.t) * a.s + c) * N : nullptr;
        float dmn = 0.0f, dmx = 0.0f;
        post_row_layer<MODE_CENTROID, 5, 4, 8>(Ld, N, dup, a.ymax, 0.0f, cur, nxt, nullptr, aout, a.force_ell, dmn, dmx);
        __syncthreads();
        fill_halo(nxt, N, h);
        __syncthreads();
        float* tmp = cur;
        cur = nxt;
        nxt = tmp;
        Ld = Lnext;
    }
    unstage_row(a.cbuf + (size_t)c * N, cur, N);
}

// Dynamic-t probe (snicit_api.cu choose_t): probe row b (one CTA each) through layers 0..tmax-1 in
// shared memory with the same layer arithmetic (Eq. 1); after every layer the row's live flag and a 64-bit
// hash of its values (+0 for -0, == semantics) go to out[l][b] (hash, live in bit 0 of a second word).
__global__ void __launch_bounds__(kCentThreads) probe_traj_kernel(PostArgs a, const float* __restrict__ rows, int tmax,
                                                                  unsigned long long* __restrict__ out) {
    extern __shared__ __align__(128) float sm[];
    __shared__ unsigned long long s_h;
    __shared__ int s_live;
    const int b = blockIdx.x;
    const int N = a.N;
    const int h = post_halo(N);
    const int dup = h == N;
    float* cur = sm;
    float* nxt = sm + N + h;
    stage_row(cur, rows + (size_t)b * N, N);
    __syncthreads();
    fill_halo(cur, N, h);
    PL Ld = load_pl(a.layers);
    for (int l = 0; l < tmax; ++l) {
        if (threadIdx.x == 0) {
            s_h = 0ull;
            s_live = 0;
        }
        __syncthreads();  // halo filled, slots reset
        const PL Lnext = load_pl(a.layers + min(l + 1, a.L - 1));
        float dmn = 0.0f, dmx = 0.0f;
        post_row_layer<MODE_CENTROID, 5, 4, 8>(Ld, N, dup, a.ymax, 0.0f, cur, nxt, nullptr, nullptr, a.force_ell, dmn,
                                               dmx);
        __syncthreads();
        unsigned long long hh = 0ull;
        int live = 0;
        for (int k = threadIdx.x; k < N; k += blockDim.x) {
            const float v = nxt[k];
            live |= v != 0.0f;
            const unsigned long long u = __float_as_uint(v + 0.0f);
            hh += (u ^ (u << 29) ^ 0x9E3779B97F4A7C15ull) * (2ull * (unsigned long long)k + 0xD1B54A32D192ED03ull);
        }
        hh = __reduce_add_sync(0xffffffffu, (unsigned)hh) | ((unsigned long long)__reduce_add_sync(0xffffffffu,
                                                                                                  (unsigned)(hh >> 32))
                                                             << 32);
        live = __any_sync(0xffffffffu, live);
        if ((threadIdx.x & 31) == 0) {
            atomicAdd(&s_h, hh);
            if (live) s_live = 1;
        }
        fill_halo(nxt, N, h);
        __syncthreads();
        if (threadIdx.x == 0) {
            out[2 * ((size_t)l * gridDim.x + b)] = s_h;
            out[2 * ((size_t)l * gridDim.x + b) + 1] = (unsigned long long)s_live;
        }
        float* tmp = cur;
        cur = nxt;
        nxt = tmp;
        Ld = Lnext;
    }
}
cudaError_t launch_probe_traj(const PostArgs& a, const float* rows, int S, int tmax, unsigned long long* out,
                              cudaStream_t st) {
    if (S <= 0 || tmax <= 0) return cudaSuccess;
    if (a.N > post_fused_max_n()) return cudaErrorInvalidValue;
    const size_t smem = sizeof(float) * 2 * (size_t)(a.N + post_halo(a.N));
    int per_sm = 1;
    cudaError_t e = blocks_per_sm((const void*)probe_traj_kernel, kCentThreads, smem, &per_sm);
    if (e != cudaSuccess) return e;
    probe_traj_kernel<<<S, kCentThreads, smem, st>>>(a, rows, tmax, out);
    return cudaGetLastError();
}

// ---- sparse-entry residue form (north_star: "only the nonzero residual entries are propagated";
// Eq. 5 / load-reduced SpMM P:860-889).  For a circulant layer, output j reads inputs (j + n nu) mod N,
// so input k feeds outputs (k - n nu) mod N, n = 0..31.  An output none of whose inputs is non-zero
// has a_r = +0 exactly (every fma adds a signed zero to +0), so Eq. 5 gives sigma((a_c + 0) + b) -
// sigma(a_c + b) == 0 (R16): only the outputs touched by a non-zero input can be non-zero, and each
// of them is evaluated with its full stored-order chain (R12; the zero taps add exact zeros), so the
// result is bit-identical to the dense-row form (tested).  A row is evaluated this way while its
// non-zero count is at most N / kSpDiv (so at most N/4 outputs are touched); otherwise densely.
constexpr int kSpDiv = 128;
__host__ __device__ inline int sp_cap(int N) { return N / kSpDiv > 0 ? N / kSpDiv : 1; }
// extra shared memory of the sparse form (ints): touched bitmap, two non-zero lists, touched list
__host__ __device__ inline int sp_ints(int N) { return (N + 31) / 32 + 2 * sp_cap(N) + 32 * sp_cap(N); }

// list the non-zero entries of row[0 .. N) into lst (first `cap` of them, in no particular order);
// returns the total count (every thread)
__device__ __forceinline__ int sp_list(const float* row, int N, int* lst, int cap, int* s_cnt) {
    const int lane = threadIdx.x & 31;
    if (threadIdx.x == 0) *s_cnt = 0;
    __syncthreads();
    for (int k0 = (threadIdx.x & ~31); k0 < N; k0 += blockDim.x) {
        const int k = k0 + lane;
        const bool nzv = k < N && row[k] != 0.0f;
        const unsigned m = __ballot_sync(0xffffffffu, nzv);
        int base = 0;
        if (lane == 0 && m) base = atomicAdd(s_cnt, __popc(m));
        base = __shfl_sync(0xffffffffu, base, 0);
        const int pos = base + __popc(m & ((1u << lane) - 1u));
        if (nzv && pos < cap) lst[pos] = k;
    }
    __syncthreads();
    return *s_cnt;
}

// One sparse-entry layer of a residue row: in (dense, non-zero exactly at lst[0 .. nnz)) -> out (all
// zero on entry; written at the touched outputs).  Returns the output's non-zero count (every thread);
// its first `cap` non-zeros are listed in lst_out.  *ntouched = outputs evaluated.
template <bool UNIF>
__device__ int sp_layer(const PL& Ld, int N, float ymax, float prune_eps, const float* __restrict__ in,
                        float* __restrict__ out, const float* __restrict__ ac, const int* lst, int nnz, int* lst_out,
                        int cap, unsigned* bm, int* tl, int* s_cnt, int* ntouched) {
    const int nu = Ld.nu, W = (N + 31) >> 5;
    const float w0 = Ld.w0, b0 = Ld.b0;
    const bool ubias = Ld.ubias != 0;
    float w[UNIF ? 1 : kPK];
    if constexpr (!UNIF) {
#pragma unroll
        for (int n = 0; n < kPK; ++n) w[n] = __ldg(Ld.wtab + n);
    }
    for (int i = threadIdx.x; i < W; i += blockDim.x) bm[i] = 0u;
    if (threadIdx.x == 0) {
        s_cnt[0] = 0;  // touched outputs
        s_cnt[1] = 0;  // non-zero outputs
    }
    __syncthreads();
    // mark the outputs fed by the non-zero inputs (32 per input)
    for (int i = threadIdx.x; i < nnz * kPK; i += blockDim.x) {
        const int k = lst[i >> 5], n = i & 31;
        int j = k - n * nu;
        j = j < 0 ? j + N : j;  // n nu < N (K nu <= N, distinct inputs)
        atomicOr(bm + (j >> 5), 1u << (j & 31));
    }
    __syncthreads();
    // touched list (per-warp scan of the bitmap words; order across warps is irrelevant)
    const int lane = threadIdx.x & 31;
    for (int i0 = (threadIdx.x & ~31); i0 < W; i0 += blockDim.x) {
        const int i = i0 + lane;
        const unsigned m = i < W ? bm[i] : 0u;
        const int c = __popc(m);
        int incl = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int v = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += v;
        }
        int base = 0;
        if (lane == 31 && incl) base = atomicAdd(&s_cnt[0], incl);
        base = __shfl_sync(0xffffffffu, base, 31);
        int pos = base + incl - c;
        for (unsigned mm = m; mm; mm &= mm - 1u) tl[pos++] = (i << 5) + __ffs(mm) - 1;
    }
    __syncthreads();
    const int nt = s_cnt[0];
    // evaluate the touched outputs: the full stored-order chain (R12), Eq. 5 epilogue
    for (int i0 = (threadIdx.x & ~31); i0 < nt; i0 += blockDim.x) {
        const int i = i0 + lane;
        float v = 0.0f;
        int j = 0;
        if (i < nt) {
            j = tl[i];
            float acc = 0.0f;
            int k = j;
#pragma unroll
            for (int n = 0; n < kPK; ++n) {
                acc = fmaf(in[k], UNIF ? w0 : w[n], acc);
                k += nu;
                k = k >= N ? k - N : k;
            }
            const float b = ubias ? b0 : __ldg(Ld.bias + j);
            v = post_epi<MODE_RESIDUAL>(acc, b, ac, j, ymax, prune_eps);
            out[j] = v;
        }
        const unsigned m = __ballot_sync(0xffffffffu, v != 0.0f);
        int base = 0;
        if (lane == 0 && m) base = atomicAdd(&s_cnt[1], __popc(m));
        base = __shfl_sync(0xffffffffu, base, 0);
        const int pos = base + __popc(m & ((1u << lane) - 1u));
        if (v != 0.0f && pos < cap) lst_out[pos] = j;
    }
    __syncthreads();
    *ntouched = nt;
    return s_cnt[1];
}

__global__ void __launch_bounds__(kPostThreads, 2) residual_traj_kernel(PostArgs a) {
    extern __shared__ __align__(128) float sm[];
    __shared__ int s_p;
    __shared__ int s_nz[3];   // per-layer non-zero count of the dense form (rotating slots)
    __shared__ int s_mn[3], s_mx[3];  // per-layer output range of the dense form (order-preserving int codes)
    __shared__ int s_cnt[3];  // sparse form: [0], [1] sp_layer's counters, [2] sp_list's (distinct slots:
                              // sp_layer may follow sp_list with no barrier in between)
    const int N = a.N;
    const int h = post_halo(N);
    const int dup = h == N;
    const int n = *a.rcount;
    const int cap = sp_cap(N);
    // three row buffers when they fit (a.smem_floats): the next residue row is loaded by the TMA engine
    // into the third while this one is processed; otherwise two and a synchronous stage
    const int nbuf = a.smem_floats >= 3 * (N + h) + (a.res_sparse ? sp_ints(N) : 0) ? 3 : 2;
    // sparse-form scratch after the row buffers
    unsigned* bm = reinterpret_cast<unsigned*>(sm + nbuf * (N + h));
    int* lsts[2] = {reinterpret_cast<int*>(bm + (N + 31) / 32), reinterpret_cast<int*>(bm + (N + 31) / 32) + cap};
    int* tl = lsts[1] + cap;
    unsigned long long c_full = 0, c_sparse = 0, c_sout = 0, c_scalar = 0;  // thread 0's work counters
    __shared__ __align__(8) uint64_t s_bar;
    __shared__ int s_next;
    int sb = 0;        // buffer receiving / holding the prefetched row
    uint32_t ph = 0;
    if (nbuf == 3 && threadIdx.x == 0) {
        mbar_init(&s_bar, 1);
        fence_proxy_async_smem();
        const int p0 = atomicAdd(a.work_counter, 1);
        s_next = p0;
        if (p0 < n) {
            mbar_arrive_expect_tx(&s_bar, (uint32_t)N * 4);
            bulk_g2s(sm, a.yhat + (size_t)a.rlist[p0] * N, (uint32_t)N * 4, &s_bar);
        }
    }
    for (;;) {
        if (nbuf == 2 && threadIdx.x == 0) s_p = atomicAdd(a.work_counter, 1);
        __syncthreads();
        const int p = nbuf == 3 ? s_next : s_p;
        if (p >= n) break;
        const int row = a.rlist[p];
        const int slot = a.cslot[row];
        float* cur;
        float* nxt;
        if (nbuf == 3) {
            cur = sm + sb * (N + h);
            nxt = sm + ((sb + 1) % 3) * (N + h);
            float* spare = sm + ((sb + 2) % 3) * (N + h);
            mbar_wait(&s_bar, ph);
            ph ^= 1u;
            __syncthreads();  // every thread past the wait before the barrier is re-armed
            if (threadIdx.x == 0) {  // the next row -> the spare buffer, behind this row's work
                const int np = atomicAdd(a.work_counter, 1);
                s_next = np;
                if (np < n) {
                    fence_proxy_async_smem();  // the spare buffer's generic accesses (previous rows) first
                    mbar_arrive_expect_tx(&s_bar, (uint32_t)N * 4);
                    bulk_g2s(spare, a.yhat + (size_t)a.rlist[np] * N, (uint32_t)N * 4, &s_bar);
                }
            }
            sb = (sb + 2) % 3;  // next row's buffer
        } else {
            cur = sm;
            nxt = sm + N + h;
            stage_row(cur, a.yhat + (size_t)row * N, N);
        }
        if (threadIdx.x < 3) {
            s_nz[threadIdx.x] = 0;
            s_mn[threadIdx.x] = 0x7fffffff;
            s_mx[threadIdx.x] = (int)0x80000000;
        }
        __syncthreads();
        fill_halo(cur, N, h);
        __syncthreads();
        bool alive = true, cst = false;
        float vr = 0.0f;
        int sc_from = a.L;  // first layer carried by a scalar
        const int cfrom = a.cfrom ? a.cfrom[slot] : a.L - a.t;
        // sparse form: nnz of `cur` and whether lsts[li] lists all of its non-zeros; nxt_zero: `nxt` is
        // all-zero in [0, N) (left so by the previous sparse layer)
        int nnz = -1, li = 0;
        bool listed = false, nxt_zero = false;
        if (a.res_sparse) {
            const int known = a.rnnz ? a.rnnz[row] : -1;  // non-zeros at t (Alg. 2's distance), if recorded
            if (known > cap) {
                nnz = known;
            } else {
                nnz = sp_list(cur, N, lsts[0], cap, &s_cnt[2]);
                listed = nnz <= cap;
            }
        }
        PL Ld = load_pl(a.layers + a.t);
        int l = a.t;
        for (; l < a.L; ++l) {
            const PL Lnext = load_pl(a.layers + min(l + 1, a.L - 1));
            const float* ac = a.a_all + ((size_t)(l - a.t) * a.s + slot) * N;
            const bool sparse = a.res_sparse && listed && Ld.kind == 1 && !a.force_ell;
            int cnt;
            bool rowconst = false;  // every output of this layer equal (dense form; a listed sparse row never is)
            float v0 = 0.0f;
            if (threadIdx.x == 0) {  // the next layer's slots (last read two barriers ago)
                s_nz[(l + 1) % 3] = 0;
                s_mn[(l + 1) % 3] = 0x7fffffff;
                s_mx[(l + 1) % 3] = (int)0x80000000;
            }
            if (sparse) {
                if (!nxt_zero)
                    for (int k = threadIdx.x; k < N; k += blockDim.x) nxt[k] = 0.0f;
                // (sp_layer's first barrier orders these stores before its own)
                int nt = 0;
                cnt = Ld.unif ? sp_layer<true>(Ld, N, a.ymax, a.prune_eps, cur, nxt, ac, lsts[li], nnz, lsts[li ^ 1],
                                               cap, bm, tl, s_cnt, &nt)
                              : sp_layer<false>(Ld, N, a.ymax, a.prune_eps, cur, nxt, ac, lsts[li], nnz,
                                                lsts[li ^ 1], cap, bm, tl, s_cnt, &nt);
                // `cur` becomes the next output buffer: clear its non-zeros (exactly lsts[li])
                for (int i = threadIdx.x; i < nnz; i += blockDim.x) cur[lsts[li][i]] = 0.0f;
                nxt_zero = true;
                li ^= 1;
                nnz = cnt;
                listed = cnt <= cap;
                if (threadIdx.x == 0) {
                    ++c_sparse;
                    c_sout += (unsigned long long)nt;
                }
            } else {
                float mn = __int_as_float(0x7f800000), mx = -__int_as_float(0x7f800000);
                const int mine = post_row_layer<MODE_RESIDUAL, 17, 16, 1>(Ld, N, dup, a.ymax, a.prune_eps, cur, nxt,
                                                                          ac, nullptr, a.force_ell, mn, mx);
                const int wsum = __reduce_add_sync(0xffffffffu, mine);
                // order-preserving integer codes of the range (bitwise-equal floats <-> equal codes)
                auto code = [](float f) {
                    const int b = __float_as_int(f);
                    return b ^ ((b >> 31) & 0x7fffffff);
                };
                const int wmn = __reduce_min_sync(0xffffffffu, code(mn)), wmx = __reduce_max_sync(0xffffffffu, code(mx));
                if ((threadIdx.x & 31) == 0) {
                    if (wsum) atomicAdd(&s_nz[l % 3], wsum);
                    atomicMin(&s_mn[l % 3], wmn);
                    atomicMax(&s_mx[l % 3], wmx);
                }
                __syncthreads();
                cnt = s_nz[l % 3];
                rowconst = s_mn[l % 3] == s_mx[l % 3];
                if (rowconst) {
                    const int c0 = s_mn[l % 3];
                    v0 = __int_as_float(c0 ^ ((c0 >> 31) & 0x7fffffff));
                }
                nxt_zero = false;
                nnz = cnt;
                listed = false;
                if (threadIdx.x == 0) ++c_full;
            }
            if (cnt == 0) {  // the residue became empty: it stays empty (R16)
                alive = false;
                break;
            }
            if (a.scalar_ok && rowconst && l + 1 < a.L && l + 1 - a.t >= cfrom) {
                // the centroid row is constant from here on (its a_c rows are) and this residue row is constant
                // too: Eq. 5 maps it to a constant row every layer -- carry it by a scalar (R25/R26; bit-identical)
                cst = true;
                vr = v0;
                ++l;
                break;
            }
            fill_halo(nxt, N, h);
            __syncthreads();
            if (a.res_sparse && !listed && nnz <= cap) {  // the dense output is sparse: list it
                nnz = sp_list(nxt, N, lsts[li], cap, &s_cnt[2]);
                listed = true;
            }
            float* tmp = cur;
            cur = nxt;
            nxt = tmp;
            Ld = Lnext;
        }
        if (cst) {  // layers l .. L-1: every thread evaluates the same scalar chain
            // the centroid's pre-activation rows are constant from here on: gather their values (one per
            // layer) into shared memory first -- the row buffers are free now -- so the serial chain does not
            // wait on one L2 round trip per layer
            float* s_acv = nxt;      // [L - l] a_c values (the row buffers are free now; not the spare one)
            float2* s_wb = reinterpret_cast<float2*>(nxt + ((a.L - l + 1) & ~1));  // [L - l] (w0, b0)
            const int nl = a.L - l;
            const bool fits = 3 * nl <= N + h;
            if (fits) {
                for (int i = threadIdx.x; i < nl; i += blockDim.x) {  // contiguous copies (acconst_kernel, load time)
                    s_acv[i] = a.acs ? a.acs[(size_t)slot * (a.L - a.t) + (l - a.t) + i]
                                     : __ldg(a.a_all + ((size_t)(l + i - a.t) * a.s + slot) * N);
                    s_wb[i] = a.wb ? a.wb[l + i] : make_float2(a.layers[l + i].w0, a.layers[l + i].b0);
                }
                __syncthreads();
            }
            const int l0 = l;
            sc_from = l;
            for (; l < a.L; ++l) {
                float w0, b0, acv;
                if (fits) {
                    const float2 wb = s_wb[l - l0];
                    w0 = wb.x;
                    b0 = wb.y;
                    acv = s_acv[l - l0];
                } else {
                    const PostLayer* pl = a.layers + l;
                    w0 = pl->w0;
                    b0 = pl->b0;
                    acv = __ldg(a.a_all + ((size_t)(l - a.t) * a.s + slot) * N);
                }
                float acc = 0.0f;
#pragma unroll
                for (int n2 = 0; n2 < kPK; ++n2) acc = fmaf(vr, w0, acc);
                float v = sigma((acv + acc) + b0, a.ymax) - sigma(acv + b0, a.ymax);
                if (a.prune_eps > 0.0f && fabsf(v) <= a.prune_eps) v = 0.0f;
                vr = v;
                if (threadIdx.x == 0) ++c_scalar;
                if (v == 0.0f) {
                    alive = false;
                    break;
                }
            }
            if (alive) {
                float4* d4 = reinterpret_cast<float4*>(a.yhat + (size_t)row * N);
                const float4 v4 = make_float4(vr, vr, vr, vr);
                for (int k = threadIdx.x; k < (N >> 2); k += blockDim.x) d4[k] = v4;
            }
        } else if (alive) {
            unstage_row(a.yhat + (size_t)row * N, cur, N);
        }
        if (threadIdx.x == 0) {
            a.ne_row[row] = alive ? 1 : 0;
            if (alive && a.alive_count) atomicAdd(a.alive_count, 1);
            if (a.dyn) {  // post layers this residue row stayed non-empty through; scalar start
                const int nl = a.L - a.t;
                atomicAdd(a.dyn + (alive ? nl : l - a.t), 1ull);
                atomicAdd(a.dyn + (nl + 1) + (cst ? sc_from - a.t : nl), 1ull);
            }
        }
        __syncthreads();  // s_p and the row buffers are reused
    }
    if (threadIdx.x == 0 && a.ctr64) {
        if (c_full) atomicAdd(a.ctr64 + C64_FULL_RL, c_full);
        if (c_sparse) atomicAdd(a.ctr64 + C64_SPARSE_RL, c_sparse);
        if (c_sout) atomicAdd(a.ctr64 + C64_SPARSE_OUT, c_sout);
        if (c_scalar) atomicAdd(a.ctr64 + C64_SCALAR_RL, c_scalar);
    }
}

// cfrom[c] = first post layer index (l - t) whose centroid pre-activation row a_c is constant (then
// every later one is: a constant input row stays constant, R25), or L - t; scans layers in order
__global__ void __launch_bounds__(256) acconst_kernel(PostArgs a) {
    const int c = blockIdx.x;
    if (c >= *a.n_cent || (a.rcount && *a.rcount == 0)) return;
    const int N = a.N, nl = a.L - a.t;
    int l2 = 0;
    if (a.cdone && a.cdone[c]) {
        l2 = 0;  // constant at t (centroid_const_kernel)
    } else {
        for (; l2 < nl; ++l2) {
            const float* row = a.a_all + ((size_t)l2 * a.s + c) * N;
            const float v0 = __ldg(row);
            bool eq = true;
            for (int k = threadIdx.x; k < N; k += blockDim.x) eq = eq && __ldg(row + k) == v0;
            if (__syncthreads_and(eq)) break;
        }
    }
    if (threadIdx.x == 0) a.cfrom[c] = l2;
    if (a.acs)  // the constant a_c values from cfrom on, contiguous per centroid (the residue rows' scalar tails)
        for (int i = l2 + threadIdx.x; i < nl; i += blockDim.x) a.acs[(size_t)c * nl + i] = __ldg(a.a_all + ((size_t)i * a.s + c) * N);
}
cudaError_t launch_acconst(const PostArgs& a, int C_max, cudaStream_t st) {
    if (C_max <= 0) return cudaSuccess;
    acconst_kernel<<<C_max, 256, 0, st>>>(a);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------ cluster version
// The centroid trajectory is a serial chain of L - t layers; one SM per centroid leaves it bound by
// a single SM's issue rate.  Here a thread-block cluster of kCL CTAs carries one centroid row: every
// layer, CTA r computes 1/kCL of the outputs and keeps them in its shared memory; the next layer's
// input window of each CTA is gathered from its peers' shared memory (distributed shared memory,
// ld through cluster-mapped addresses), and one cluster barrier per layer orders the exchange.
// Output ownership per layer: index partition (CTA r owns outputs [r*S, (r+1)*S), S = N/kCL) for
// nu == 1 and general strides, residue partition (CTA r owns residues [r*nu/kCL, (r+1)*nu/kCL) at
// all 32 a) for Q == 32 layers, so every CTA's input window is a small, mostly local set.
constexpr int kCL = 8;
constexpr int kClThreads = 512;
constexpr int kClMaxWin = 16384;  // floats of the gathered input window

__device__ __forceinline__ int ilog2(int x) { return 31 - __clz(x); }

__global__ void __cluster_dims__(kCL, 1, 1) __launch_bounds__(kClThreads) centroid_cluster_kernel(PostArgs a) {
    extern __shared__ __align__(128) float sm[];
    __shared__ float* s_rbase[2][kCL];  // peers' slice buffers (cluster-mapped generic pointers)
    // constant-row detection (R25 from the layer the row becomes constant): each CTA's output range
    // (bits of sigma outputs, >= 0) pushed to every rank before the layer's cluster barrier
    __shared__ unsigned s_vmn[2][kCL], s_vmx[2][kCL];
    __shared__ unsigned s_bmn[2], s_bmx[2];
    __shared__ unsigned* s_vbase[2][kCL];
    cg::cluster_group cl = cg::this_cluster();
    const int r = (int)cl.block_rank();
    const int cid = blockIdx.x / kCL;
    const int C = *a.n_cent;
    if (cid >= C || (a.cdone && a.cdone[cid])) return;  // uniform over the cluster
    const bool want_a = a.a_all && (!a.rcount || *a.rcount > 0);  // a_c rows only for residue rows
    const int N = a.N, S = N / kCL;  // powers of two (centroid_cluster_ok)
    const int shS = ilog2(S);
    float* slice[2] = {sm, sm + S};
    float* win = sm + 2 * S;
    if (threadIdx.x < 2 * kCL) {
        const int bsel = threadIdx.x / kCL, o = threadIdx.x % kCL;
        s_rbase[bsel][o] = cl.map_shared_rank(slice[bsel], o);
        s_vbase[bsel][o] = cl.map_shared_rank(bsel ? &s_vmx[0][0] : &s_vmn[0][0], o);
    }
    for (int i = threadIdx.x; i < S; i += blockDim.x) slice[0][i] = a.cbuf[(size_t)cid * N + r * S + i];
    int prev_part = 0, prev_nu = 1, cur = 0;
    bool cst = false;
    float vc = 0.0f;
    int lc = a.L;
    cl.sync();
    PL Ld = load_pl(a.layers + a.t);
    for (int l = a.t; l < a.L; ++l) {
        const int par = (l - a.t) & 1;
        if (threadIdx.x == 0) {
            s_bmn[par] = 0xffffffffu;
            s_bmx[par] = 0u;
        }
        unsigned umn = 0xffffffffu, umx = 0u;
        const PL Lnext = load_pl(a.layers + min(l + 1, a.L - 1));
        const int nu = Ld.nu, cls = Ld.cls;
        const int shnu = ilog2(nu), Q = N >> shnu;
        const int part = cls == PCLS_Q32 ? 1 : 0;
        const float w0 = Ld.w0, b0 = Ld.b0;
        const bool ubias = Ld.ubias != 0, unif = Ld.unif != 0;
        const float* __restrict__ bias = Ld.bias;
        float wr[kPK];
        if (unif) {
#pragma unroll
            for (int n = 0; n < kPK; ++n) wr[n] = w0;
        } else {
#pragma unroll
            for (int n = 0; n < kPK; ++n) wr[n] = __ldg(Ld.wtab + n);
        }
        float* aout = want_a ? a.a_all + ((size_t)(l - a.t) * a.s + cid) * N : nullptr;
        // ---- gather this CTA's input window from the peers' slices (previous layer's outputs)
        float* const* rb = s_rbase[cur];
        const int shnp = ilog2(prev_nu);
        const int shcp = prev_part ? shnp - 3 : 0;  // log2(prev_nu / kCL)
        auto fetch = [&](int k) -> float {           // element k of the previous layer's row
            int o, off;
            if (prev_part == 0) {
                o = k >> shS;
                off = k & (S - 1);
            } else {
                const int aa = k >> shnp, c = k & (prev_nu - 1);
                o = c >> shcp;
                off = (aa << shcp) | (c & ((1 << shcp) - 1));
            }
            return rb[o][off];
        };
        int q0 = 0, a_s = 0, c0 = 0, cs = 0, shcs = 0;
        if (cls == PCLS_NU1) {
            q0 = r * S;
            // S + 40 >= the last item's window end (a0 + M + 31 with a0 < S, M = 5)
            for (int i = threadIdx.x; i < S + 40; i += blockDim.x) win[i] = fetch((q0 + i) & (N - 1));
        } else if (cls == PCLS_GEN) {
            a_s = r * (S >> shnu);
            const int wlen = ((S >> shnu) + kPK) << shnu;
            for (int i = threadIdx.x; i < wlen; i += blockDim.x) {
                const int aa = i >> shnu, c = i & (nu - 1);
                win[i] = fetch((((a_s + aa) & (Q - 1)) << shnu) | c);
            }
        } else {
            shcs = shnu - 3;
            cs = nu >> 3;
            c0 = r * cs;
            for (int i = threadIdx.x; i < (32 << shcs); i += blockDim.x) {
                const int aa = i >> shcs, cc = i & (cs - 1);
                win[i] = fetch((aa << shnu) + c0 + cc);
            }
        }
        __syncthreads();
        // ---- compute this CTA's outputs (stored-order fma chains, R12) into its next slice
        float* out = slice[cur ^ 1];
        auto emit = [&](float acc, int q, int so) {
            const float b = ubias ? b0 : __ldg(bias + q);
            if (aout) aout[q] = acc;
            const float o = sigma(acc + b, a.ymax);
            out[so] = o;
            const unsigned u = __float_as_uint(o + 0.0f);
            umn = min(umn, u);
            umx = max(umx, u);
        };
        if (cls == PCLS_NU1) {
            constexpr int M = 5, WIN = M + kPK - 1;  // odd M: conflict-free window loads
            for (int it = threadIdx.x; it * M < S; it += blockDim.x) {
                const int a0 = it * M;
                float R[WIN];
#pragma unroll
                for (int i = 0; i < WIN; ++i) R[i] = win[a0 + i];
#pragma unroll
                for (int m = 0; m < M; ++m) {
                    if (a0 + m < S) {
                        float acc = 0.0f;
#pragma unroll
                        for (int n = 0; n < kPK; ++n) acc = fmaf(R[m + n], wr[n], acc);
                        emit(acc, q0 + a0 + m, a0 + m);
                    }
                }
            }
        } else if (cls == PCLS_GEN) {
            constexpr int M = 4, WIN = M + kPK - 1;
            const int na = S >> shnu;
            for (int it = threadIdx.x; it < nu * ((na + M - 1) / M); it += blockDim.x) {
                const int c = it & (nu - 1), al = (it >> shnu) * M;
                float R[WIN];
#pragma unroll
                for (int i = 0; i < WIN; ++i) R[i] = win[((al + i) << shnu) + c];
#pragma unroll
                for (int m = 0; m < M; ++m) {
                    if (al + m < na) {
                        float acc = 0.0f;
#pragma unroll
                        for (int n = 0; n < kPK; ++n) acc = fmaf(R[m + n], wr[n], acc);
                        emit(acc, ((a_s + al + m) << shnu) + c, ((al + m) << shnu) + c);
                    }
                }
            }
        } else {
            constexpr int OG = 4;
            for (int it = threadIdx.x; it < cs * (32 / OG); it += blockDim.x) {
                const int cc = it & (cs - 1), g0 = (it >> shcs) * OG;
                float R[32];
#pragma unroll
                for (int j = 0; j < 32; ++j) R[j] = win[(((g0 + j) & 31) << shcs) + cc];
#pragma unroll
                for (int mm = 0; mm < OG; ++mm) {
                    float acc = 0.0f;
#pragma unroll
                    for (int n = 0; n < kPK; ++n) acc = fmaf(R[(mm + n) & 31], wr[n], acc);
                    emit(acc, ((g0 + mm) << shnu) + c0 + cc, ((g0 + mm) << shcs) + cc);
                }
            }
        }
        if (a.scalar_ok) {  // this CTA's output range -> every rank
            umn = __reduce_min_sync(0xffffffffu, umn);
            umx = __reduce_max_sync(0xffffffffu, umx);
            if ((threadIdx.x & 31) == 0) {
                atomicMin(&s_bmn[par], umn);
                atomicMax(&s_bmx[par], umx);
            }
            __syncthreads();
            if (threadIdx.x < kCL) {
                s_vbase[0][threadIdx.x][par * kCL + r] = s_bmn[par];
                s_vbase[1][threadIdx.x][par * kCL + r] = s_bmx[par];
            }
        }
        cl.sync();  // outputs (and ranges) of this layer visible cluster-wide; nobody still reads slice[cur]
        cur ^= 1;
        prev_part = part;
        prev_nu = nu;
        Ld = Lnext;
        if (a.scalar_ok) {
            unsigned gmn = 0xffffffffu, gmx = 0u;
#pragma unroll
            for (int o = 0; o < kCL; ++o) {
                gmn = min(gmn, s_vmn[par][o]);
                gmx = max(gmx, s_vmx[par][o]);
            }
            if (gmn == gmx && l + 1 < a.L) {  // the row is the constant v: every later layer maps it to a
                cst = true;                   // constant row (one weight, one bias, R25)
                vc = __uint_as_float(gmn);
                lc = l + 1;
                break;
            }
        }
    }
    if (cst) {  // layers lc .. L-1 by one scalar chain; a_c rows (constant) written when residues need them
        // the slice / window buffers are free now: (w0, b0) of the remaining layers, gathered in parallel,
        // then the serial chain (memoised on (v, w0): SDGC repeats one weight and reaches a fixed point),
        // then the a_c rows written by all threads
        const int nl = a.L - lc;
        float2* s_wb2 = reinterpret_cast<float2*>(sm);
        float* s_ac = reinterpret_cast<float*>(s_wb2 + nl);
        const bool fits = 3 * nl <= a.smem_floats;
        __shared__ float s_vfin;
        if (fits) {
            __syncthreads();  // every thread is past its reads of the buffers
            for (int i = threadIdx.x; i < nl; i += blockDim.x) {
                const PostLayer* pl = a.layers + lc + i;
                s_wb2[i] = make_float2(pl->w0, pl->b0);
            }
            __syncthreads();
            if (threadIdx.x == 0) {
                float v = vc, pv = 0.0f, pw = 0.0f, pacc = 0.0f;
                bool have = false;
                for (int i = 0; i < nl; ++i) {
                    const float2 wb = s_wb2[i];
                    float acc;
                    if (have && __float_as_uint(v) == __float_as_uint(pv) && __float_as_uint(wb.x) == __float_as_uint(pw)) {
                        acc = pacc;
                    } else {
                        acc = 0.0f;
#pragma unroll
                        for (int n = 0; n < kPK; ++n) acc = fmaf(v, wb.x, acc);
                        pv = v;
                        pw = wb.x;
                        pacc = acc;
                        have = true;
                    }
                    s_ac[i] = acc;
                    v = sigma(acc + wb.y, a.ymax);
                }
                s_vfin = v;
            }
            __syncthreads();
            if (want_a)
                for (int i = 0; i < nl; ++i) {
                    float* dst = a.a_all + ((size_t)(lc + i - a.t) * a.s + cid) * N + r * S;
                    const float acc = s_ac[i];
                    for (int j = threadIdx.x; j < S; j += blockDim.x) dst[j] = acc;
                }
            vc = s_vfin;
        } else {
            for (int l = lc; l < a.L; ++l) {
                const PostLayer* pl = a.layers + l;
                const float w0 = pl->w0, b0 = pl->b0;
                float acc = 0.0f;
#pragma unroll
                for (int n = 0; n < kPK; ++n) acc = fmaf(vc, w0, acc);
                if (want_a) {
                    float* dst = a.a_all + ((size_t)(l - a.t) * a.s + cid) * N + r * S;
                    for (int i = threadIdx.x; i < S; i += blockDim.x) dst[i] = acc;
                }
                vc = sigma(acc + b0, a.ymax);
            }
        }
        for (int i = threadIdx.x; i < S; i += blockDim.x) a.cbuf[(size_t)cid * N + r * S + i] = vc;
        return;
    }
    // ---- the final centroid row back to global memory
    for (int i = threadIdx.x; i < S; i += blockDim.x) {
        int k;
        if (prev_part == 0) {
            k = r * S + i;
        } else {
            const int csz = prev_nu / kCL;
            const int aa = i / csz, cc = i - aa * csz;
            k = aa * prev_nu + r * csz + cc;
        }
        a.cbuf[(size_t)cid * N + k] = slice[cur][i];
    }
}

// host: can the cluster kernel carry layers [t, L)?  (every layer circulant, partition-compatible)
static bool pow2(int x) { return x > 0 && (x & (x - 1)) == 0; }
bool centroid_cluster_ok(int N, const int* nu, const int* cls, int t, int L) {
    if (!pow2(N) || N < kCL * 64) return false;  // shift/mask index arithmetic
    const int S = N / kCL;
    for (int l = t; l < L; ++l) {
        if (cls[l] < 0 || !pow2(nu[l])) return false;  // not circulant (or ELL forced)
        if (cls[l] == PCLS_NU1) {
            if (S + 40 > kClMaxWin) return false;
        } else if (cls[l] == PCLS_Q32) {
            if (nu[l] % kCL != 0) return false;
        } else {
            if (S % nu[l] != 0 || (size_t)(S / nu[l] + kPK) * nu[l] > kClMaxWin) return false;
        }
    }
    return true;
}

// ------------------------------------------------------------------ constant centroid rows
// A circulant layer with uniform bias maps a constant row (every element bitwise equal to v) to a
// constant row: every output j evaluates the same stored-order chain acc = fma(v, w_n, acc),
// n = 0..K-1, then sigma(acc + b) -- the chain of Eq. 1 / Eq. 5 (first case) with all inputs equal
// (R12).  So a centroid that is constant at t is carried through the post layers (all circulant,
// uniform weights and bias; checked by the caller) by one scalar chain per layer, bit-identical to
// the full-row evaluation (tested against the oracle and the general kernels).  Each CTA checks one
// centroid row (bitwise AND == OR), preloads the layers' (w0, b0) into shared memory, runs the scalar
// trajectory in one thread, then writes the final row (and a_c of every layer when residues need it).
__global__ void __launch_bounds__(256) centroid_const_kernel(PostArgs a, float* cout, int* cdone, int* ndone) {
    extern __shared__ float2 s_wb[];  // [L - t] (w0, b0); then acc per layer (a_all)
    __shared__ unsigned s_and[8], s_or[8];
    __shared__ float s_v;
    const int c = blockIdx.x;
    if (c >= *a.n_cent) return;
    const int N = a.N, nl = a.L - a.t;
    const float* row = a.cbuf + (size_t)c * N;
    unsigned an = 0xffffffffu, o = 0u;
    for (int j = threadIdx.x; j < N; j += blockDim.x) {
        const unsigned u = __float_as_uint(row[j]);
        an &= u;
        o |= u;
    }
    for (int d = 16; d; d >>= 1) {
        an &= __shfl_xor_sync(0xffffffffu, an, d);
        o |= __shfl_xor_sync(0xffffffffu, o, d);
    }
    if ((threadIdx.x & 31) == 0) {
        s_and[threadIdx.x >> 5] = an;
        s_or[threadIdx.x >> 5] = o;
    }
    for (int l = threadIdx.x; l < nl; l += blockDim.x) {
        const PostLayer* p = a.layers + a.t + l;
        s_wb[l] = make_float2(p->w0, p->b0);
    }
    __syncthreads();
    an = s_and[0];
    o = s_or[0];
    for (int w = 1; w < (int)(blockDim.x >> 5); ++w) {
        an &= s_and[w];
        o |= s_or[w];
    }
    if (an != o) {  // not constant: the general trajectory kernels carry it
        if (threadIdx.x == 0) cdone[c] = 0;
        return;
    }
    float* s_acc = reinterpret_cast<float*>(s_wb + nl);
    // Fixed-point prefix, evaluated in parallel: layer l maps the constant v0 to itself (bitwise) for every
    // l < lfix, so by induction the row enters each of those layers as v0 (acc_l = chain(v0, w_l)) and
    // leaves the prefix as v0; the serial chain below starts at lfix (SDGC: YMAX is a fixed point of every
    // layer, so lfix = L - t and nothing is serial)
    __shared__ int s_lfix;
    const float v0 = __uint_as_float(an);
    if (threadIdx.x == 0) s_lfix = nl;
    __syncthreads();
    for (int l = threadIdx.x; l < nl; l += blockDim.x) {
        const float2 wb = s_wb[l];
        float acc = 0.0f;
#pragma unroll
        for (int n = 0; n < kPK; ++n) acc = fmaf(v0, wb.x, acc);
        s_acc[l] = acc;
        if (__float_as_uint(sigma(acc + wb.y, a.ymax)) != an) atomicMin(&s_lfix, l);
    }
    __syncthreads();
    const int lfix = s_lfix;
    if (threadIdx.x == 0) {
        float v = v0;
        // the chain is a pure function of (v, w0): reuse the previous layer's value when both repeat
        float pv = 0.0f, pw = 0.0f, pacc = 0.0f;
        bool have = false;
        for (int l = lfix; l < nl; ++l) {
            const float2 wb = s_wb[l];
            float acc;
            if (have && __float_as_uint(v) == __float_as_uint(pv) && __float_as_uint(wb.x) == __float_as_uint(pw)) {
                acc = pacc;
            } else {
                acc = 0.0f;
#pragma unroll
                for (int n = 0; n < kPK; ++n) acc = fmaf(v, wb.x, acc);
                pv = v;
                pw = wb.x;
                pacc = acc;
                have = true;
            }
            s_acc[l] = acc;
            v = sigma(acc + wb.y, a.ymax);
        }
        s_v = v;
    }
    __syncthreads();
    if (a.a_all && (!a.rcount || *a.rcount > 0))  // a_c rows only when residue rows need them
        for (int l = 0; l < nl; ++l) {
            float* dst = a.a_all + ((size_t)l * a.s + c) * N;
            const float acc = s_acc[l];
            for (int j = threadIdx.x; j < N; j += blockDim.x) dst[j] = acc;
        }
    const float v = s_v;
    for (int j = threadIdx.x; j < N; j += blockDim.x) cout[(size_t)c * N + j] = v;
    if (threadIdx.x == 0) {
        cdone[c] = 1;
        atomicAdd(ndone, 1);
    }
}

cudaError_t launch_centroid_const(const PostArgs& a, float* cout, int* cdone, int* ndone, int C_max, cudaStream_t st) {
    if (C_max <= 0) return cudaSuccess;
    const size_t smem = (size_t)(a.L - a.t) * (sizeof(float2) + sizeof(float));
    int per_sm = 1;
    cudaError_t e = blocks_per_sm((const void*)centroid_const_kernel, 256, smem, &per_sm);
    if (e != cudaSuccess) return e;
    centroid_const_kernel<<<C_max, 256, smem, st>>>(a, cout, cdone, ndone);
    return cudaGetLastError();
}

cudaError_t launch_centroid_cluster(const PostArgs& a_in, int C_max, int win_max, cudaStream_t st) {
    if (C_max <= 0) return cudaSuccess;
    PostArgs a = a_in;
    const size_t smem = sizeof(float) * (2 * (size_t)(a.N / kCL) + (size_t)win_max);
    a.smem_floats = (int)(smem / sizeof(float));
    int per_sm = 1;
    cudaError_t e = blocks_per_sm((const void*)centroid_cluster_kernel, kClThreads, smem, &per_sm);
    if (e != cudaSuccess) return e;
    centroid_cluster_kernel<<<C_max * kCL, kClThreads, smem, st>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_centroid_traj(const PostArgs& a, int C_max, cudaStream_t st) {
    if (C_max <= 0) return cudaSuccess;
    const size_t smem = sizeof(float) * 2 * (size_t)(a.N + post_halo(a.N));
    int per_sm = 1;
    cudaError_t e = blocks_per_sm((const void*)centroid_traj_kernel, kCentThreads, smem, &per_sm);
    if (e != cudaSuccess) return e;
    centroid_traj_kernel<<<C_max, kCentThreads, smem, st>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_residual_traj(const PostArgs& a_in, int max_rows, int num_sms, cudaStream_t st) {
    if (max_rows <= 0) return cudaSuccess;
    PostArgs a = a_in;
    const size_t row = sizeof(float) * (size_t)(a.N + post_halo(a.N));
    const size_t sp = sizeof(int) * (size_t)sp_ints(a.N);
    const size_t lim = (size_t)220 * 1024;
    size_t smem = 2 * row;
    if (a.res_sparse && smem + sp <= lim)
        smem += sp;
    else
        a.res_sparse = 0;
    if (smem + row <= lim) smem += row;  // a third row buffer: the next row is prefetched
    a.smem_floats = (int)(smem / sizeof(float));
    int per_sm = 1;
    cudaError_t e = blocks_per_sm((const void*)residual_traj_kernel, kPostThreads, smem, &per_sm);
    if (e != cudaSuccess) return e;
    int grid = num_sms * per_sm;
    if (grid > max_rows) grid = max_rows;
    residual_traj_kernel<<<grid, kPostThreads, smem, st>>>(a);
    return cudaGetLastError();
}

}  // namespace snicit
