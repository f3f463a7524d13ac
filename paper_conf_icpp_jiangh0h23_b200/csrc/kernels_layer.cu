// kernels_layer.cu -- the fused sparse layer kernels of the SNICIT hot path (sm_100a).
//
// One launch computes, for every active row r of the list and every output neuron j,
//   acc = fma-chain over the stored order of column j  (Eq. 1; R12)
// and one of three epilogues (LayerMode):
//   PLAIN     y'[j] = sigma(acc + b[j])                                  (Eq. 1)
//   CENTROID  y'[j] = sigma(acc + b[j]), and a_c[j] = acc kept           (Eq. 5 first case)
//   RESIDUAL  y'[j] = sigma((a_c[j] + acc) + b[j]) - sigma(a_c[j] + b[j]) (Eq. 5 second case,
//             Alg. 3 line 9); optional near-zero pruning
// plus the per-row "any non-zero" flag consumed by row compaction (ne_rec, Alg. 3 lines 10-13).
//
// This file: layer_ell_kernel (the circulant fast path is in kernels_circ.cu)
//  * layer_ell_kernel: general CSC stored as n-major ELL (uint16 or int32 indices); a tile of RT
//    rows in shared memory (TMA), one thread per output column, RT accumulators in registers so
//    each index/value load is reused RT times.  N too large for shared memory: rows gathered from
//    global memory (L1/L2).
#include <cuda_runtime.h>

#include <cstdlib>
#include <map>
#include <mutex>
#include <utility>

#include "snicit_internal.cuh"

namespace snicit {

// Blocks per SM of a kernel at a given dynamic shared-memory size, cached per (device, kernel, smem)
// so a launch costs no host-side attribute/occupancy queries after the first (the post-convergence
// loop launches ~2 kernels per layer for up to 1890 layers).
cudaError_t blocks_per_sm(const void* kern, int threads, size_t smem, int* out) {
    static std::mutex mu;
    static std::map<std::pair<std::pair<int, const void*>, size_t>, int> cache;
    static std::map<std::pair<int, const void*>, size_t> attr;  // max dynamic smem set per kernel
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    const auto key = std::make_pair(std::make_pair(dev, kern), smem);
    {
        std::lock_guard<std::mutex> g(mu);
        auto it = cache.find(key);
        if (it != cache.end()) {
            *out = it->second;
            return cudaSuccess;
        }
        // the attribute is a per-kernel maximum: only ever raise it (a kernel launched with several
        // shared-memory sizes must keep the largest one allowed)
        size_t& cur = attr[key.first];
        if (smem > cur) {
            e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            if (e != cudaSuccess) return e;
            cur = smem;
        }
    }
    int per_sm = 1;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, threads, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) per_sm = 1;
    std::lock_guard<std::mutex> g(mu);
    cache[key] = per_sm;
    *out = per_sm;
    return cudaSuccess;
}

constexpr int kEllThreads = 512;

// ------------------------------------------------------------------------------ ELL (general)
constexpr int kEllSurvCap = 256;
// block-wide: append the buffered surviving rows to the next active list (one atomic per batch)
__device__ __forceinline__ void ell_flush(const LayerArgs& a, const int* s_surv, int* s_nsurv, int* s_pos) {
    __syncthreads();
    const int n = *s_nsurv;
    if (n > 0) {
        if (threadIdx.x == 0) *s_pos = atomicAdd(a.app_count, n);
        __syncthreads();
        const int pos = *s_pos;
        for (int i = threadIdx.x; i < n; i += blockDim.x) a.app_list[pos + i] = s_surv[i];
    }
    __syncthreads();
    if (threadIdx.x == 0) *s_nsurv = 0;
    __syncthreads();
}
template <int MODE, int RT, bool IDX16, bool UNIF, bool RAGGED, bool SMEM>
__global__ void __launch_bounds__(kEllThreads, 1) layer_ell_kernel(LayerArgs a) {
    extern __shared__ __align__(128) unsigned char smem[];
    const int N = a.N;
    float* s_in = reinterpret_cast<float*>(smem);
    uint64_t* bar = reinterpret_cast<uint64_t*>(s_in + (SMEM ? (size_t)RT * N : 0));
    int* s_flag = reinterpret_cast<int*>(bar + 1);
    int* s_row = s_flag + RT;
    int* s_slot = s_row + RT;
    int* s_surv = s_slot + RT;  // kEllSurvCap surviving row ids (fused dead-row compaction)
    __shared__ int s_nsurv, s_pos;
    __shared__ unsigned s_cmn[RT], s_cmx[RT];  // constant-row mode: each row's output range (bits)

    if (blockIdx.x == 0 && threadIdx.x == 0 && a.zero_count) *a.zero_count = 0;
    if (threadIdx.x == 0) s_nsurv = 0;
    const int count = *a.count;
    const int ntiles = (count + RT - 1) / RT;
    if (SMEM && threadIdx.x == 0) {
        mbar_init(bar, 1);
        fence_proxy_async_smem();
    }
    __syncthreads();
    uint32_t parity = 0;
    for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const int r0 = tile * RT;
        const int nr = min(RT, count - r0);
        if (threadIdx.x < RT) {
            const int row = a.rows[r0 + min((int)threadIdx.x, nr - 1)];
            s_row[threadIdx.x] = row;
            s_flag[threadIdx.x] = 0;
            s_cmn[threadIdx.x] = 0xffffffffu;
            s_cmx[threadIdx.x] = 0u;
            if constexpr (MODE == MODE_RESIDUAL) s_slot[threadIdx.x] = a.cslot[row];
        }
        __syncthreads();
        if constexpr (SMEM) {
            if (threadIdx.x == 0) {
                mbar_arrive_expect_tx(bar, (uint32_t)(nr * N * 4));
                for (int i = 0; i < nr; ++i)
                    bulk_g2s(s_in + (size_t)i * N, a.yin + (size_t)s_row[i] * N, N * 4, bar);
            }
            mbar_wait(bar, parity);
            parity ^= 1u;
        }
        const float* base[RT];
#pragma unroll
        for (int r = 0; r < RT; ++r)
            base[r] = SMEM ? (s_in + (size_t)(r < nr ? r : 0) * N) : (a.yin + (size_t)s_row[r] * N);
        int anyr = 0;  // bit r: row r has a non-zero output in this thread's columns
        unsigned rmn[RT], rmx[RT];  // constant-row mode: this thread's output range per row
#pragma unroll
        for (int r = 0; r < RT; ++r) {
            rmn[r] = 0xffffffffu;
            rmx[r] = 0u;
        }
        for (int j = threadIdx.x; j < N; j += blockDim.x) {
            const int len = RAGGED ? (int)a.len[j] : a.K;
            float acc[RT];
#pragma unroll
            for (int r = 0; r < RT; ++r) acc[r] = 0.0f;
#pragma unroll 4
            for (int n = 0; n < len; ++n) {
                const size_t e = (size_t)n * N + j;
                const int k = IDX16 ? (int)__ldg(a.idx16 + e) : __ldg(a.idx32 + e);
                const float w = UNIF ? a.w0 : __ldg(a.val + e);
#pragma unroll
                for (int r = 0; r < RT; ++r) acc[r] = fmaf(base[r][k], w, acc[r]);
            }
#pragma unroll
            for (int r = 0; r < RT; ++r) {
                if (r < nr) {
                    const int row = s_row[r];
                    const float v = epilogue<MODE>(a, acc[r], __ldg(a.bias + j), j, row, MODE == MODE_RESIDUAL ? s_slot[r] : 0);
                    a.yout[(size_t)row * N + j] = v;
                    if (v != 0.0f) anyr |= 1 << r;
                    if (MODE == MODE_PLAIN) {
                        const unsigned u = __float_as_uint(v + 0.0f);
                        rmn[r] = min(rmn[r], u);
                        rmx[r] = max(rmx[r], u);
                    }
                }
            }
        }
#pragma unroll
        for (int r = 0; r < RT; ++r)
            if (anyr & (1 << r)) s_flag[r] = 1;
        if (MODE == MODE_PLAIN && a.cmin) {  // constant-row mode (R26): each row's range over the tile's outputs
#pragma unroll
            for (int r = 0; r < RT; ++r) {
                const unsigned wmn = __reduce_min_sync(0xffffffffu, rmn[r]), wmx = __reduce_max_sync(0xffffffffu, rmx[r]);
                if ((threadIdx.x & 31) == 0) {
                    atomicMin(&s_cmn[r], wmn);
                    atomicMax(&s_cmx[r], wmx);
                }
            }
        }
        __syncthreads();
        if (threadIdx.x < nr) {
            const uint8_t f = s_flag[threadIdx.x] ? 1 : 0;
            if (a.flag_pos) a.flag_pos[r0 + threadIdx.x] = f;
            if (a.flag_row) a.flag_row[s_row[threadIdx.x]] = f;
            if (MODE == MODE_PLAIN && a.cmin) {  // the tile holds whole rows: the range is final
                a.cmin[r0 + threadIdx.x] = s_cmn[threadIdx.x];
                a.cmax[r0 + threadIdx.x] = s_cmx[threadIdx.x];
            }
        }
        if (a.app_list && threadIdx.x == 0) {
            for (int i = 0; i < nr; ++i)
                if (s_flag[i]) s_surv[s_nsurv++] = s_row[i];
        }
        __syncthreads();
        if (a.app_list && s_nsurv > kEllSurvCap - RT) ell_flush(a, s_surv, &s_nsurv, &s_pos);
    }
    if (a.app_list) ell_flush(a, s_surv, &s_nsurv, &s_pos);
}

// ---- row-interleaved variant (the general-CSC hot path): the RT rows of a tile are stored
// interleaved, element (k, r) at k RT + r, so one thread (output column j) fetches input k of all RT rows
// with one 16-byte shared load (RT = 4) or two (RT = 8) instead of RT scattered 4-byte loads, and feeds
// them to packed FFMA2 pairs (rows r, r + 1).  For RT = 8 the two 16-byte halves of input k are stored
// in the order h0 = (k >> 2) & 1 first, so the first load of a warp touches chunk (2k + h0) mod 8 -- all
// eight 16-byte bank groups -- instead of only the even ones.  Rows are loaded with coalesced float4
// global loads and transposed on the shared-memory store; the next tile's rows are prefetched into L2.
template <int RT>
__device__ __forceinline__ int il_pos(int k, int r) {
    if constexpr (RT == 8) {
        const int h0 = (k >> 2) & 1;
        return k * 8 + (((r >> 2) ^ h0) << 2) + (r & 3);
    } else {
        return k * RT + r;
    }
}

// RT = 4 tiles (64 KB at N = 4096) run 256 threads at three CTAs per SM (other CTAs cover a tile's load);
// RT = 8 / 2: 512 threads, one CTA per SM
template <int RT>
constexpr int kIlThreads = RT == 4 ? 256 : kEllThreads;
template <int RT>
constexpr int kIlMinBlocks = RT == 4 ? 3 : 1;

template <int MODE, int RT, bool IDX16, bool UNIF, bool RAGGED>
__global__ void __launch_bounds__(kIlThreads<RT>, kIlMinBlocks<RT>) layer_ell_il_kernel(LayerArgs a) {
    static_assert(RT == 2 || RT == 4 || RT == 8, "RT");
    extern __shared__ __align__(128) unsigned char smem[];
    const int N = a.N;
    float* s_in = reinterpret_cast<float*>(smem);
    int* s_flag = reinterpret_cast<int*>(s_in + (size_t)RT * N);
    int* s_row = s_flag + RT;
    int* s_slot = s_row + RT;
    int* s_surv = s_slot + RT;  // kEllSurvCap surviving row ids (fused dead-row compaction)
    __shared__ int s_nsurv, s_pos;
    __shared__ unsigned s_cmn[RT], s_cmx[RT];  // constant-row mode: each row's output range (bits)

    if (blockIdx.x == 0 && threadIdx.x == 0 && a.zero_count) *a.zero_count = 0;
    if (threadIdx.x == 0) s_nsurv = 0;
    const int count = *a.count;
    const int ntiles = (count + RT - 1) / RT;
    const int N4 = N >> 2;
    __syncthreads();
    for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const int r0 = tile * RT;
        const int nr = min(RT, count - r0);
        if (threadIdx.x < RT) {
            const int row = a.rows[r0 + min((int)threadIdx.x, nr - 1)];
            s_row[threadIdx.x] = row;
            s_flag[threadIdx.x] = 0;
            s_cmn[threadIdx.x] = 0xffffffffu;
            s_cmx[threadIdx.x] = 0u;
            if constexpr (MODE == MODE_RESIDUAL) s_slot[threadIdx.x] = a.cslot[row];
        } else if (threadIdx.x < 2 * RT) {  // the next tile's rows -> L2 while this one computes
            const int nt = tile + gridDim.x, i = threadIdx.x - RT;
            if (nt < ntiles && nt * RT + i < count)
                bulk_prefetch_l2(a.yin + (size_t)a.rows[nt * RT + i] * N, (uint32_t)N * 4);
        }
        __syncthreads();
        // transposed load: thread -> (row r, float4 chunk c)
        for (int t = threadIdx.x; t < RT * N4; t += blockDim.x) {
            const int r = t % RT, c = t / RT;
            const float4 v = __ldg(reinterpret_cast<const float4*>(a.yin + (size_t)s_row[r] * N) + c);
            s_in[il_pos<RT>(4 * c + 0, r)] = v.x;
            s_in[il_pos<RT>(4 * c + 1, r)] = v.y;
            s_in[il_pos<RT>(4 * c + 2, r)] = v.z;
            s_in[il_pos<RT>(4 * c + 3, r)] = v.w;
        }
        __syncthreads();
        int anyr = 0;  // bit r: row r has a non-zero output in this thread's columns
        unsigned rmn[RT], rmx[RT];  // constant-row mode: this thread's output range per row (bits, +0 for -0)
#pragma unroll
        for (int r = 0; r < RT; ++r) {
            rmn[r] = 0xffffffffu;
            rmx[r] = 0u;
        }
        for (int j = threadIdx.x; j < N; j += blockDim.x) {
            const int len = RAGGED ? (int)a.len[j] : a.K;
            unsigned long long acc[RT / 2];
#pragma unroll
            for (int q = 0; q < RT / 2; ++q) acc[q] = 0ull;
#pragma unroll 4
            for (int n = 0; n < len; ++n) {
                const size_t e = (size_t)n * N + j;
                const int k = IDX16 ? (int)__ldg(a.idx16 + e) : __ldg(a.idx32 + e);
                const float w = UNIF ? a.w0 : __ldg(a.val + e);
                const unsigned long long W2 = f2_pack(w, w);
                if constexpr (RT == 8) {
                    const int h0 = (k >> 2) & 1;
                    const float4 lo = *reinterpret_cast<const float4*>(s_in + k * 8 + (h0 << 2));        // rows 0..3
                    const float4 hi = *reinterpret_cast<const float4*>(s_in + k * 8 + ((h0 ^ 1) << 2));  // rows 4..7
                    acc[0] = f2_fma(f2_pack(lo.x, lo.y), W2, acc[0]);
                    acc[1] = f2_fma(f2_pack(lo.z, lo.w), W2, acc[1]);
                    acc[2] = f2_fma(f2_pack(hi.x, hi.y), W2, acc[2]);
                    acc[3] = f2_fma(f2_pack(hi.z, hi.w), W2, acc[3]);
                } else if constexpr (RT == 4) {
                    const float4 v = *reinterpret_cast<const float4*>(s_in + k * 4);
                    acc[0] = f2_fma(f2_pack(v.x, v.y), W2, acc[0]);
                    acc[1] = f2_fma(f2_pack(v.z, v.w), W2, acc[1]);
                } else {
                    const float2 v = *reinterpret_cast<const float2*>(s_in + k * 2);
                    acc[0] = f2_fma(f2_pack(v.x, v.y), W2, acc[0]);
                }
            }
            const float bj = __ldg(a.bias + j);
#pragma unroll
            for (int q = 0; q < RT / 2; ++q) {
                float z[2];
                f2_unpack(acc[q], z[0], z[1]);
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const int r = 2 * q + h;
                    if (r < nr) {
                        const int row = s_row[r];
                        const float v = epilogue<MODE>(a, z[h], bj, j, row, MODE == MODE_RESIDUAL ? s_slot[r] : 0);
                        a.yout[(size_t)row * N + j] = v;
                        if (v != 0.0f) anyr |= 1 << r;
                        if (MODE == MODE_PLAIN) {
                            const unsigned u = __float_as_uint(v + 0.0f);
                            rmn[r] = min(rmn[r], u);
                            rmx[r] = max(rmx[r], u);
                        }
                    }
                }
            }
        }
#pragma unroll
        for (int r = 0; r < RT; ++r)
            if (anyr & (1 << r)) s_flag[r] = 1;
        if (MODE == MODE_PLAIN && a.cmin) {  // constant-row mode (R26): each row's range over the tile's outputs
#pragma unroll
            for (int r = 0; r < RT; ++r) {
                const unsigned wmn = __reduce_min_sync(0xffffffffu, rmn[r]), wmx = __reduce_max_sync(0xffffffffu, rmx[r]);
                if ((threadIdx.x & 31) == 0) {
                    atomicMin(&s_cmn[r], wmn);
                    atomicMax(&s_cmx[r], wmx);
                }
            }
        }
        __syncthreads();
        if (threadIdx.x < nr) {
            const uint8_t f = s_flag[threadIdx.x] ? 1 : 0;
            if (a.flag_pos) a.flag_pos[r0 + threadIdx.x] = f;
            if (a.flag_row) a.flag_row[s_row[threadIdx.x]] = f;
            if (MODE == MODE_PLAIN && a.cmin) {  // the tile holds whole rows: the range is final
                a.cmin[r0 + threadIdx.x] = s_cmn[threadIdx.x];
                a.cmax[r0 + threadIdx.x] = s_cmx[threadIdx.x];
            }
        }
        if (a.app_list && threadIdx.x == 0) {
            for (int i = 0; i < nr; ++i)
                if (s_flag[i]) s_surv[s_nsurv++] = s_row[i];
        }
        __syncthreads();
        if (a.app_list && s_nsurv > kEllSurvCap - RT) ell_flush(a, s_surv, &s_nsurv, &s_pos);
    }
    if (a.app_list) ell_flush(a, s_surv, &s_nsurv, &s_pos);
}

bool ell_smem_ok(int N) { return (size_t)N * 4 * 2 <= 200 * 1024 && N % 4 == 0; }

template <int MODE, int RT, bool SMEM>
static cudaError_t launch_ell_t(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st) {
    const size_t smem = (SMEM ? (size_t)RT * a.N * 4 : 0) + 16 + 12 * RT + 16 + 4 * kEllSurvCap;
    const bool i16 = a.idx16 != nullptr, unif = a.val == nullptr, rag = a.len != nullptr;
    void (*kern)(LayerArgs) = nullptr;
    constexpr bool IL = SMEM && (RT == 2 || RT == 4 || RT == 8);  // row-interleaved tile
#define SNICIT_PICK(I, U, G)                                                                 \
    if (i16 == I && unif == U && rag == G) {                                                 \
        if constexpr (IL)                                                                    \
            kern = layer_ell_il_kernel<MODE, (IL ? RT : 2), I, U, G>;                        \
        else                                                                                 \
            kern = layer_ell_kernel<MODE, RT, I, U, G, SMEM>;                                \
    }
    SNICIT_PICK(true, true, false)
    SNICIT_PICK(true, false, false)
    SNICIT_PICK(true, true, true)
    SNICIT_PICK(true, false, true)
    SNICIT_PICK(false, true, false)
    SNICIT_PICK(false, false, false)
    SNICIT_PICK(false, true, true)
    SNICIT_PICK(false, false, true)
#undef SNICIT_PICK
    int per_sm = 1;
    const int threads = IL ? kIlThreads<RT> : kEllThreads;
    cudaError_t e = blocks_per_sm((const void*)kern, threads, smem, &per_sm);
    if (e != cudaSuccess) return e;
    const int tiles = (max_rows + RT - 1) / RT;
    int grid = num_sms * per_sm;
    if (grid > tiles) grid = tiles;
    if (grid < 1) grid = 1;
    kern<<<grid, threads, smem, st>>>(a);
    return cudaGetLastError();
}

template <int MODE>
static cudaError_t launch_ell_m(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st) {
    if (!ell_smem_ok(a.N)) return launch_ell_t<MODE, 4, false>(a, max_rows, num_sms, st);
    const size_t row = (size_t)a.N * 4;
    static const int force_rt = [] {
        const char* e = getenv("SNICIT_ELL_RT");  // A/B experiments only
        return e ? atoi(e) : 0;
    }();
    if (force_rt == 4 && max_rows >= 4 && 4 * row <= 70 * 1024) return launch_ell_t<MODE, 4, true>(a, max_rows, num_sms, st);
    if (max_rows >= 8 && 8 * row <= 200 * 1024) return launch_ell_t<MODE, 8, true>(a, max_rows, num_sms, st);
    if (max_rows >= 4 && 4 * row <= 200 * 1024) return launch_ell_t<MODE, 4, true>(a, max_rows, num_sms, st);
    if (max_rows >= 2 && 2 * row <= 200 * 1024) return launch_ell_t<MODE, 2, true>(a, max_rows, num_sms, st);
    return launch_ell_t<MODE, 1, true>(a, max_rows, num_sms, st);
}

bool gen_enabled() {
    static const bool on = [] {
        const char* e = getenv("SNICIT_GEN");  // "0": the previous ELL kernels (A/B experiments only)
        return !(e && e[0] == '0');
    }();
    return on;
}

cudaError_t launch_layer_ell(const LayerArgs& a, int mode, int max_rows, int num_sms, cudaStream_t st) {
    if (max_rows <= 0) return cudaSuccess;
    // few rows (the centroid rows of the post phase): the tiled kernel would occupy a handful of CTAs, the
    // thread-per-output kernel below spreads them over more (C5: 128 centroid rows per post layer)
    if (a.gidx && gen_enabled() && max_rows > 256) return launch_layer_gen(a, mode, max_rows, num_sms, st);
    switch (mode) {
        case MODE_PLAIN: return launch_ell_m<MODE_PLAIN>(a, max_rows, num_sms, st);
        case MODE_CENTROID: return launch_ell_m<MODE_CENTROID>(a, max_rows, num_sms, st);
        default: return launch_ell_m<MODE_RESIDUAL>(a, max_rows, num_sms, st);
    }
}

}  // namespace snicit
