// kernels_convert.cu -- row compaction, cluster-based conversion and recovery kernels (sm_100a).
//
//  compact_kernel       ne_idx from ne_rec on device, order-preserving
//  downsample_kernel    column sampling + sum downsampling (Sec. 3.2.1, Fig. 3a)
//  prune_kernel         sample pruning, Alg. 1 with Eq. 2 (reading R2), then the
//                       centroid list y*
//  map_residual_kernel  mapper M (Eq. 3) and residue errors (Eq. 4),
//                       Alg. 2
//  recover_kernel       final results recovery (Eq. 6) + category flags (R13)
#include <cuda_runtime.h>
#include <string.h>

#include "snicit_internal.cuh"

namespace snicit {

__global__ void iota_kernel(int* out, int n, int* count_out) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) out[i] = i;
    if (count_out && blockIdx.x == 0 && threadIdx.x == 0) *count_out = n;
}
cudaError_t launch_iota(int* out, int n, int* count_out, cudaStream_t st) {
    int grid = n > 0 ? (n + 255) / 256 : 1;
    if (grid > 4096) grid = 4096;
    iota_kernel<<<grid, 256, 0, st>>>(out, n, count_out);
    return cudaGetLastError();
}

__global__ void fill_i32_kernel(int* out, int n, int v) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) out[i] = v;
}
cudaError_t launch_fill_i32(int* out, int n, int v, cudaStream_t st) {
    if (n <= 0) return cudaSuccess;
    int grid = (n + 255) / 256;
    if (grid > 4096) grid = 4096;
    fill_i32_kernel<<<grid, 256, 0, st>>>(out, n, v);
    return cudaGetLastError();
}
__global__ void fill_u8_kernel(uint8_t* out, int n, uint8_t v) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) out[i] = v;
}
cudaError_t launch_fill_u8(uint8_t* out, int n, uint8_t v, cudaStream_t st) {
    if (n <= 0) return cudaSuccess;
    int grid = (n + 255) / 256;
    if (grid > 4096) grid = 4096;
    fill_u8_kernel<<<grid, 256, 0, st>>>(out, n, v);
    return cudaGetLastError();
}

// flag_row[rows[p]] = 1 for p < *count
__global__ void mark_rows_kernel(const int* rows, const int* count, uint8_t* flag_row) {
    const int n = *count;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) flag_row[rows[i]] = 1;
}
cudaError_t launch_mark_rows(const int* rows, const int* count, uint8_t* flag_row, int max_rows, cudaStream_t st) {
    int grid = max_rows > 0 ? (max_rows + 255) / 256 : 1;
    if (grid > 4096) grid = 4096;
    mark_rows_kernel<<<grid, 256, 0, st>>>(rows, count, flag_row);
    return cudaGetLastError();
}

// One warp per listed row: flag_pos[p] = any_k y[rows[p]][k] != 0.
__global__ void row_nonzero_kernel(const float* __restrict__ y, int N, const int* rows, const int* count,
                                   uint8_t* flag_pos) {
    const int n = *count;
    const int lane = threadIdx.x & 31;
    const int warps = (gridDim.x * blockDim.x) >> 5;
    for (int p = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; p < n; p += warps) {
        const float* r = y + (size_t)rows[p] * N;
        int any = 0;
        for (int k = lane; k < N; k += 32) any |= (r[k] != 0.0f);
        any = __any_sync(0xffffffffu, any);
        if (lane == 0) flag_pos[p] = any ? 1 : 0;
    }
}
cudaError_t launch_row_nonzero(const float* y, int N, const int* rows, const int* count, uint8_t* flag_pos,
                               int max_rows, int num_sms, cudaStream_t st) {
    int grid = (max_rows + 7) / 8;
    if (grid > num_sms * 8) grid = num_sms * 8;
    if (grid < 1) grid = 1;
    row_nonzero_kernel<<<grid, 256, 0, st>>>(y, N, rows, count, flag_pos);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------ compaction
// Order-preserving stream compaction (ne_idx "sorted indices of ne_rec == true", rebuilt
// on device instead of the paper's serial host loop):
//   out = [list_in[i] for i < *count_in if flag_pos[i]]      (list_in NULL: the identity)
// Two launches over chunks of kChunk positions: per-chunk counts, then each chunk sums the counts
// before it (<= a few hundred), scans its own flags (16 per thread, 16-byte loads) and scatters.
constexpr int kCompactThreads = 256;
constexpr int kChunk = kCompactThreads * 16;

__device__ __forceinline__ int popc_bytes(uint4 v) {
    // number of non-zero bytes among 16
    int c = 0;
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const uint32_t x = w[i];
        const uint32_t nz = ((x & 0x7f7f7f7fu) + 0x7f7f7f7fu | x) & 0x80808080u;  // high bit per non-zero byte
        c += __popc(nz);
    }
    return c;
}

__device__ __forceinline__ uint4 load_flags16(const uint8_t* f, int base, int n) {
    if (base + 16 <= n && (reinterpret_cast<uintptr_t>(f + base) & 15) == 0)
        return *reinterpret_cast<const uint4*>(f + base);
    uint8_t b[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) b[i] = (base + i < n) ? f[base + i] : 0;
    uint4 v;
    memcpy(&v, b, 16);
    return v;
}

__global__ void __launch_bounds__(kCompactThreads) compact_count_kernel(const int* count_in,
                                                                        const uint8_t* __restrict__ flag_pos,
                                                                        int* block_counts) {
    const int n = *count_in;
    const int base = blockIdx.x * kChunk + threadIdx.x * 16;
    int c = base < n ? popc_bytes(load_flags16(flag_pos, base, n)) : 0;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) c += __shfl_down_sync(0xffffffffu, c, o);
    __shared__ int ws[kCompactThreads / 32];
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = c;
    __syncthreads();
    if (threadIdx.x == 0) {
        int t = 0;
        for (int w = 0; w < kCompactThreads / 32; ++w) t += ws[w];
        block_counts[blockIdx.x] = t;
    }
}

__global__ void __launch_bounds__(kCompactThreads) compact_scatter_kernel(const int* __restrict__ list_in,
                                                                          const int* count_in,
                                                                          uint8_t* __restrict__ flag_pos,
                                                                          const int* block_counts,
                                                                          int* __restrict__ list_out,
                                                                          int* count_out, int clear,
                                                                          uint8_t* __restrict__ row_flags) {
    const int n = *count_in;
    const int nblk = (n + kChunk - 1) / kChunk;
    __shared__ int s_prefix, s_ws[kCompactThreads / 32];
    if ((int)blockIdx.x >= max(nblk, 1)) return;
    if (threadIdx.x < 32) {  // exclusive prefix of the chunks before this one
        int p = 0;
        for (int b = threadIdx.x; b < (int)blockIdx.x; b += 32) p += block_counts[b];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) p += __shfl_down_sync(0xffffffffu, p, o);
        if (threadIdx.x == 0) s_prefix = p;
    }
    const int base = blockIdx.x * kChunk + threadIdx.x * 16;
    const uint4 v = base < n ? load_flags16(flag_pos, base, n) : make_uint4(0, 0, 0, 0);
    const int c = popc_bytes(v);
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    int incl = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
    }
    if (lane == 31) s_ws[wid] = incl;
    __syncthreads();
    int woff = 0, total = 0;
    for (int w = 0; w < kCompactThreads / 32; ++w) {
        const int t = s_ws[w];
        if (w < wid) woff += t;
        total += t;
    }
    int pos = s_prefix + woff + incl - c;
    uint8_t bytes[16];
    memcpy(bytes, &v, 16);
#pragma unroll
    for (int i = 0; i < 16; ++i) {
        if (base + i >= n) break;
        const int id = list_in ? list_in[base + i] : base + i;
        if (bytes[i]) list_out[pos++] = id;
        if (row_flags) row_flags[id] = bytes[i] ? 1 : 0;  // e.g. ne_rec of residue rows (Alg. 3 l.13)
        if (clear) flag_pos[base + i] = 0;                 // flags OR-ed by several CTAs start at 0
    }
    if ((int)blockIdx.x == max(nblk, 1) - 1 && threadIdx.x == 0) *count_out = s_prefix + total;
}

cudaError_t launch_compact(const int* list_in, const int* count_in, const uint8_t* flag_pos, int* list_out,
                           int* count_out, int max_n, int* scratch, cudaStream_t st, int clear,
                           uint8_t* row_flags) {
    const int nblk = max(1, (max_n + kChunk - 1) / kChunk);
    compact_count_kernel<<<nblk, kCompactThreads, 0, st>>>(count_in, flag_pos, scratch);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    compact_scatter_kernel<<<nblk, kCompactThreads, 0, st>>>(list_in, count_in, const_cast<uint8_t*>(flag_pos),
                                                              scratch, list_out, count_out, clear, row_flags);
    return cudaGetLastError();
}
int compact_scratch_ints(int max_n) { return max(1, (max_n + kChunk - 1) / kChunk); }

// ------------------------------------------------------------------------------ conversion
// Sum downsampling: block (g, q) sums segment g of sampled row q ("first s columns", of
// the live list, R14) in fp64 (R3).  Segments of floor(N/n), last takes the remainder (R15).
__global__ void downsample_kernel(const float* __restrict__ y, int N, const int* rows, const int* count, int s,
                                  int n, double* F) {
    const int q = blockIdx.y;
    const int s_eff = min(s, *count);
    if (q >= s_eff) return;
    const int g = blockIdx.x;
    const int seg = N / n;
    const int k0 = g * seg, k1 = (g == n - 1) ? N : k0 + seg;
    const float* r = y + (size_t)rows[q] * N;
    double sum = 0.0;
    for (int k = k0 + threadIdx.x; k < k1; k += blockDim.x) sum += (double)r[k];
    __shared__ double red[32];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) sum += __shfl_down_sync(0xffffffffu, sum, o);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = sum;
    __syncthreads();
    if (threadIdx.x < 32) {
        double v = (threadIdx.x < (blockDim.x >> 5)) ? red[threadIdx.x] : 0.0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
        if (threadIdx.x == 0) F[(size_t)g * s + q] = v;
    }
}
cudaError_t launch_downsample(const float* y, int N, const int* rows, const int* count, int s, int n_seg,
                              double* F, cudaStream_t st) {
    const int n = n_seg <= 0 ? N : n_seg;
    const int seg = N / n;
    const int threads = seg >= 256 ? 256 : (seg >= 64 ? 64 : 32);
    dim3 grid(n, s);
    downsample_kernel<<<grid, threads, 0, st>>>(y, N, rows, count, s, n, F);
    return cudaGetLastError();
}

// Alg. 1 in one CTA (P:603-605 launches <<<1,(n,s)>>>; here threads loop over the n x s pairs so
// any n*s works, R5).  diff counts are integer atomics in shared memory: order-independent and
// deterministic.  After the loop the survivors (ascending position = ascending row id, since the
// live list is ascending) form y*; cent_cnt = |y*|.
constexpr int kPruneThreads = 1024;
__global__ void __launch_bounds__(kPruneThreads) prune_kernel(const double* __restrict__ F, const int* count, int s,
                                                              int n, float eta, float eps, const int* rows,
                                                              int* cent, int* n_cent, int* s_eff_out,
                                                              int* col_idx) {
    extern __shared__ int sh[];
    int* tmp_idx = sh;     // [s]
    int* diff = sh + s;    // [s]
    const int s_eff = min(s, *count);
    for (int q = threadIdx.x; q < s_eff; q += blockDim.x) tmp_idx[q] = q;  // lines 3-4
    const double thr = (double)n * (double)eps;
    const double eta_d = (double)eta;
    for (int cmp = 0; cmp < s_eff; ++cmp) {  // line 6
        __syncthreads();
        if (tmp_idx[cmp] == -1) continue;    // line 7 (uniform: read after the barrier)
        for (int q = threadIdx.x; q < s_eff; q += blockDim.x) diff[q] = 0;  // lines 10-11
        __syncthreads();
        for (int p = threadIdx.x; p < n * s_eff; p += blockDim.x) {         // lines 13-14, Eq. 2
            const int g = p / s_eff, q = p - g * s_eff;
            if (q != cmp && tmp_idx[q] != -1) {
                const double d = fabs(F[(size_t)g * s + q] - F[(size_t)g * s + cmp]);
                if (d > eta_d) atomicAdd(&diff[q], 1);
            }
        }
        __syncthreads();
        for (int q = threadIdx.x; q < s_eff; q += blockDim.x)                // lines 16-17
            if (q != cmp && tmp_idx[q] != -1 && (double)diff[q] < thr) tmp_idx[q] = -1;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        int C = 0;
        for (int q = 0; q < s_eff; ++q) {
            col_idx[q] = tmp_idx[q];
            if (tmp_idx[q] != -1) cent[C++] = rows[q];
        }
        *n_cent = C;
        *s_eff_out = s_eff;
    }
}
cudaError_t launch_prune(const double* F, const int* count, int s, int n_seg, float eta, float eps,
                         const int* rows, int* cent, int* n_cent, int* s_eff, int* col_idx, cudaStream_t st) {
    const size_t smem = 2 * sizeof(int) * (size_t)s;
    prune_kernel<<<1, kPruneThreads, smem, st>>>(F, count, s, n_seg, eta, eps, rows, cent, n_cent, s_eff, col_idx);
    return cudaGetLastError();
}

// Alg. 2 / Eq. 3-4: one CTA per live row.  L0 distance to each centroid (element-wise '!=' counts,
// Alg. 2 lines 10-12), first minimum over ascending y* wins (strict '<', R6).  Centroid rows are
// copied to the compact centroid buffer (slot = position in y*), M = -1 and ne = 1 (R7); mapped
// rows get M = centroid row id, ne = (dist != 0), and their residue Y_r - Y_c written only if ne.
constexpr int kMapThreads = 256;
__global__ void __launch_bounds__(kMapThreads) map_residual_kernel(const float* __restrict__ y, int N,
                                                                   const int* rows, const int* count,
                                                                   const int* cent, const int* n_cent, int* M,
                                                                   int* cslot, uint8_t* ne_row, uint8_t* flag_pos,
                                                                   float* __restrict__ yhat,
                                                                   float* __restrict__ cbuf,
                                                                   const uint8_t* __restrict__ rconst,
                                                                   const float* __restrict__ rval,
                                                                   unsigned long long* nnz_sum) {
    __shared__ int red[kMapThreads / 32];
    __shared__ int s_best, s_slot;
    const int n = *count;
    const int C = *n_cent;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int N4 = N >> 2;
    for (int p = blockIdx.x; p < n; p += gridDim.x) {
        const int r = rows[p];
        const float4* y4 = reinterpret_cast<const float4*>(y + (size_t)r * N);
        if (threadIdx.x == 0) {
            s_slot = -1;
            for (int c = 0; c < C; ++c)
                if (cent[c] == r) s_slot = c;
        }
        __syncthreads();
        const int slot = s_slot;
        if (slot >= 0) {  // centroid row (Eq. 4 second case)
            float4* d4 = reinterpret_cast<float4*>(cbuf + (size_t)slot * N);
            for (int k = threadIdx.x; k < N4; k += blockDim.x) d4[k] = y4[k];
            if (threadIdx.x == 0) {
                M[r] = -1;
                cslot[r] = slot;
                ne_row[r] = 1;
                flag_pos[p] = 0;
            }
            __syncthreads();
            continue;
        }
        if (rconst && rconst[r]) {
            // constant row (R26, flags from the pre phase): its L0 distance to a centroid that is the
            // same constant is 0 and to any other centroid > 0, so the first such centroid is Alg. 2's
            // argmin (strict <) -- empty residue, nothing to read or write
            int hit = -1;
            const float v = rval[r];
            for (int c = 0; c < C && hit < 0; ++c)
                if (rconst[cent[c]] && rval[cent[c]] == v) hit = c;
            if (hit >= 0) {
                if (threadIdx.x == 0) {
                    M[r] = cent[hit];
                    cslot[r] = hit;
                    ne_row[r] = 0;
                    flag_pos[p] = 0;
                }
                continue;  // uniform across the CTA: no barrier needed
            }
        }
        int best_dist = N + 1, best = 0;  // Alg. 2 line 3 (tracked by thread 0)
        for (int c = 0; c < C; ++c) {
            const float4* c4 = reinterpret_cast<const float4*>(y + (size_t)cent[c] * N);
            int cnt = 0;
            for (int k = threadIdx.x; k < N4; k += blockDim.x) {
                const float4 a = y4[k], b = c4[k];
                cnt += (a.x != b.x) + (a.y != b.y) + (a.z != b.z) + (a.w != b.w);
            }
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) cnt += __shfl_down_sync(0xffffffffu, cnt, o);
            if (lane == 0) red[wid] = cnt;
            __syncthreads();
            if (threadIdx.x == 0) {
                int d = 0;
                for (int w = 0; w < kMapThreads / 32; ++w) d += red[w];
                if (d < best_dist) {  // lines 14-16
                    best_dist = d;
                    best = c;
                }
            }
            __syncthreads();
        }
        if (threadIdx.x == 0) {
            s_best = best;
            s_slot = best_dist;  // reuse as the distance broadcast
            M[r] = cent[best];   // line 25
            cslot[r] = best;
            const uint8_t ne = best_dist != 0 ? 1 : 0;  // lines 26-29
            ne_row[r] = ne;
            flag_pos[p] = ne;
            // the residue's non-zeros are exactly the differing elements (x - y != 0 <=> x != y, finite)
            if (nnz_sum && ne) atomicAdd(nnz_sum, (unsigned long long)best_dist);
        }
        __syncthreads();
        if (s_slot != 0) {  // residue only needed for non-empty rows (Eq. 4 first case)
            const float4* c4 = reinterpret_cast<const float4*>(y + (size_t)cent[s_best] * N);
            float4* o4 = reinterpret_cast<float4*>(yhat + (size_t)r * N);
            for (int k = threadIdx.x; k < N4; k += blockDim.x) {
                const float4 a = y4[k], b = c4[k];
                o4[k] = make_float4(a.x - b.x, a.y - b.y, a.z - b.z, a.w - b.w);
            }
        }
        __syncthreads();
    }
}
cudaError_t launch_map_residual(const float* y, int N, const int* rows, const int* count, const int* cent,
                                const int* n_cent, int* M, int* cslot, uint8_t* ne_row, uint8_t* flag_pos,
                                float* yhat, float* cbuf, int max_rows, int num_sms, cudaStream_t st,
                                const uint8_t* rconst, const float* rval, unsigned long long* nnz_sum) {
    int grid = num_sms * 8;
    if (grid > max_rows) grid = max_rows;
    if (grid < 1) grid = 1;
    map_residual_kernel<<<grid, kMapThreads, 0, st>>>(y, N, rows, count, cent, n_cent, M, cslot, ne_row, flag_pos,
                                                      yhat, cbuf, rconst, rval, nnz_sum);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------ recovery
// Eq. 6: Y_r = Yhat_r (centroid); (ne ? Yhat_r : 0) + Yhat_M(r) (mapped, R18); 0 (dead, R23).
// plain != 0 (t >= L): Y_r = live ? yfinal_r : 0.  cat[r] = any non-zero (R13).  One CTA per row.
constexpr int kRecThreads = 256;
__global__ void __launch_bounds__(kRecThreads) recover_kernel(int N, int R, int plain,
                                                              const float* __restrict__ yfinal,
                                                              const uint8_t* live_row, const int* M,
                                                              const int* cslot, const uint8_t* ne_row,
                                                              const float* __restrict__ cbuf,
                                                              float* __restrict__ y_out, uint8_t* cat,
                                                              int dead_zeroed) {
    const int N4 = N >> 2;
    for (int r = blockIdx.x; r < R; r += gridDim.x) {
        int mode;  // 0 zero, 1 copy a, 2 a + c, 3 0 + c
        const float4* a4 = nullptr;
        const float4* c4 = nullptr;
        if (plain) {
            mode = live_row[r] ? 1 : 0;
            a4 = reinterpret_cast<const float4*>(yfinal + (size_t)r * N);
        } else {
            const int m = M[r];
            if (m == -2) {
                mode = 0;
            } else if (m == -1) {
                mode = 1;
                a4 = reinterpret_cast<const float4*>(cbuf + (size_t)cslot[r] * N);
            } else {
                c4 = reinterpret_cast<const float4*>(cbuf + (size_t)cslot[r] * N);
                if (ne_row[r]) {
                    mode = 2;
                    a4 = reinterpret_cast<const float4*>(yfinal + (size_t)r * N);
                } else {
                    mode = 3;
                }
            }
        }
        if (mode == 0 && dead_zeroed) {  // dead row: y_out already zeroed by the pre phase
            if (threadIdx.x == 0) cat[r] = 0;
            continue;  // uniform across the CTA
        }
        int any = 0;
        float4* o4 = y_out ? reinterpret_cast<float4*>(y_out + (size_t)r * N) : nullptr;
        for (int k = threadIdx.x; k < N4; k += blockDim.x) {
            float4 v;
            if (mode == 0) {
                v = make_float4(0.f, 0.f, 0.f, 0.f);
            } else if (mode == 1) {
                v = a4[k];
            } else if (mode == 2) {
                const float4 a = a4[k], c = c4[k];
                v = make_float4(a.x + c.x, a.y + c.y, a.z + c.z, a.w + c.w);
            } else {
                const float4 c = c4[k];
                v = make_float4(0.0f + c.x, 0.0f + c.y, 0.0f + c.z, 0.0f + c.w);
            }
            any |= (v.x != 0.f) | (v.y != 0.f) | (v.z != 0.f) | (v.w != 0.f);
            if (o4) o4[k] = v;
        }
        any = __syncthreads_or(any);
        if (threadIdx.x == 0) cat[r] = any ? 1 : 0;
    }
}
cudaError_t launch_recover(int N, int R, int plain, const float* yfinal, const uint8_t* live_row, const int* M,
                           const int* cslot, const uint8_t* ne_row, const float* cbuf, float* y_out,
                           uint8_t* cat, int num_sms, cudaStream_t st, int dead_zeroed) {
    if (R <= 0) return cudaSuccess;
    int grid = num_sms * 8;
    if (grid > R) grid = R;
    recover_kernel<<<grid, kRecThreads, 0, st>>>(N, R, plain, yfinal, live_row, M, cslot, ne_row, cbuf, y_out,
                                                 cat, dead_zeroed);
    return cudaGetLastError();
}

// ------------------------------------------------------------------ packed binary input (snicit_infer_packed)
// One thread per 4 consecutive outputs of a row: coalesced float4 stores; the 8 threads sharing a
// 32-bit word read it from L1.  N % 4 == 0 (load-time requirement), W = ceil(N / 32) words per row.
__global__ void unpack_bits_kernel(const uint32_t* __restrict__ bits, long long quads, int N, int W, float one,
                                   float* __restrict__ y) {
    const int qpr = N >> 2;
    for (long long q = (long long)blockIdx.x * blockDim.x + threadIdx.x; q < quads;
         q += (long long)gridDim.x * blockDim.x) {
        const long long r = q / qpr;
        const int j = (int)(q - r * qpr) << 2;
        const uint32_t w = __ldg(bits + r * W + (j >> 5)) >> (j & 31);
        float4 v;
        v.x = (w & 1u) ? one : 0.0f;
        v.y = (w & 2u) ? one : 0.0f;
        v.z = (w & 4u) ? one : 0.0f;
        v.w = (w & 8u) ? one : 0.0f;
        reinterpret_cast<float4*>(y + r * N)[j >> 2] = v;
    }
}

cudaError_t launch_unpack_bits(const uint32_t* bits, int R, int N, float one, float* y, int num_sms, cudaStream_t st) {
    const long long quads = (long long)R * (N / 4);
    if (quads <= 0) return cudaSuccess;
    long long grid = (quads + 255) / 256;
    if (grid > (long long)num_sms * 16) grid = (long long)num_sms * 16;
    unpack_bits_kernel<<<(int)grid, 256, 0, st>>>(bits, quads, N, (N + 31) / 32, one, y);
    return cudaGetLastError();
}

// Category export (multi-GPU all-gather): out[0] = total (int64), out[1 + i] = offset +
// catlist[i] for i < min(total, cap) -- device to device, no host synchronisation
__global__ void export_categories_kernel(const int* __restrict__ catlist, const int* __restrict__ count,
                                         long long offset, long long* __restrict__ out, long long cap) {
    const long long n = *count;
    const long long m = n < cap ? n : cap;
    if (blockIdx.x == 0 && threadIdx.x == 0) out[0] = n;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (long long)gridDim.x * blockDim.x)
        out[1 + i] = offset + catlist[i];
}
cudaError_t launch_export_categories(const int* catlist, const int* count, long long offset, long long* out,
                                     long long cap, cudaStream_t st) {
    long long grid = (cap + 255) / 256;
    if (grid > 1024) grid = 1024;
    if (grid < 1) grid = 1;
    export_categories_kernel<<<(int)grid, 256, 0, st>>>(catlist, count, offset, out, cap);
    return cudaGetLastError();
}

}  // namespace snicit
