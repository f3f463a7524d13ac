// kernels_circ_seg.cu -- circulant layer kernel for large rows (N >= ~8K: C3 = 16384, C4 = 65536).
//
// Same arithmetic as kernels_circ.cu (the stored-order fma chain of every output, reading R12), but a
// row no longer has to fit in shared memory: a tile is (row, segment) of about 4K outputs.
//   A-segment (nu == 1, or a general stride whose staged window is small): outputs a in [a_s, a_e)
//     (all residues c); the stage holds a-rows [a_s, a_e + 31) mod Q, i.e. the contiguous float range
//     [a_s*nu, (a_e + 31)*nu) mod N (one or two TMA bulk copies), so windows never wrap.
//   C-segment (Q == 32, or a general stride with small Q): outputs for residues c in [c_s, c_s + C_T)
//     and every a; the stage holds a-rows 0 .. Q + 31 (the first 31 repeated for Q > 32 windows)
//     of C_T contiguous floats each: one bulk copy per a-row, issued by all producer lanes.
// The stage element (a_local, c_local) lives at a_local * P + c_local (P = nu for A-segments, C_T
// for C-segments), outputs are written back in place and TMA-stored (one copy for A-segments, one per
// a-row for C-segments).  A row's any-non-zero flag is OR-ed into flag_pos[list position] from every
// segment (plain stores of 1; the ordered compaction that reads it also clears it).
//
// Pipeline: as kernels_circ.cu -- one producer warp (S stages, row ids via the tile index) and 8
// consumer warps (one work item per thread), mbarrier full/empty handshakes, no CTA-wide barriers.
#include <cuda_runtime.h>

#include "snicit_internal.cuh"

namespace snicit {

constexpr int kSegThreads = 256;
constexpr int kSK = 32;
constexpr int kSegMaxStages = 6;

struct SegGeom {
    int cseg;      // 0: A-segment, 1: C-segment
    int cls;       // 0: nu == 1 (M = 17), 1: Q == 32 (whole class), 2: general (M = 16)
    int nseg;      // segments per row
    int A_T;       // A: a-rows of outputs per segment
    int C_T;       // C: residues per segment
    int P;         // stage pitch (floats per staged a-row)
    int rows_st;   // staged a-rows per segment
    int stage;     // floats per stage (16-byte multiple)
    int items;     // work items per (full) segment
};

__host__ __device__ inline int seg_M(int cls) { return cls == 0 ? 17 : (cls == 1 ? 32 : 16); }

static SegGeom seg_geom(int N, int nu) {
    SegGeom g{};
    const int Q = N / nu;
    g.cls = nu == 1 ? 0 : (Q == 32 ? 1 : 2);
    const int M = seg_M(g.cls);
    if (g.cls == 0) {  // A-segments of 256 items x 17 outputs
        g.cseg = 0;
        g.A_T = 256 * M;
        g.P = 1;
        g.rows_st = g.A_T + kSK;  // + 31-row halo, rounded so every copy is a 16-byte multiple
        g.items = 256;
    } else if (g.cls == 2 && (size_t)(256 / nu * M + kSK - 1) * nu <= 8192 && nu <= 256) {
        g.cseg = 0;  // general stride, A-segments: nu residues x (A_T / 16) chunks = 256 items
        g.A_T = (256 / nu) * M;
        g.P = nu;
        g.rows_st = g.A_T + kSK;
        g.items = 256;
    } else {
        g.cseg = 1;  // C-segments: C_T residues; Q32: one item per residue, general: Q/16 per residue
        const int per_c = g.cls == 1 ? 1 : (Q + M - 1) / M;
        g.C_T = 256 / per_c;
        if (g.C_T > nu) g.C_T = nu;
        g.C_T &= ~3;  // 16-byte rows
        if (g.C_T < 4) g.C_T = 4;
        g.P = g.C_T;
        g.rows_st = g.cls == 1 ? 32 : Q + kSK - 1;
        g.items = g.C_T * per_c;
    }
    if (g.cseg == 0) {
        const int Aall = Q;
        g.nseg = (Aall + g.A_T - 1) / g.A_T;
    } else {
        g.nseg = (nu + g.C_T - 1) / g.C_T;
    }
    g.stage = ((g.rows_st * g.P) + 3) & ~3;
    return g;
}

bool circ_seg_supported(int N, int K, int nu) {
    if (K != kSK || nu <= 0 || N % nu != 0 || N % 4 != 0) return false;
    if ((long long)K * nu > N) return false;
    const SegGeom g = seg_geom(N, nu);
    if (g.cseg == 1 && (nu % 4 != 0 || g.C_T < 4)) return false;
    if (g.cseg == 0 && g.cls == 2 && (nu % 4 != 0)) return false;
    return (size_t)g.stage * 4 * 2 <= 200 * 1024;
}

template <int MODE, bool UNIF, bool UBIAS>
__global__ void __launch_bounds__(kSegThreads + 32, 2) layer_circ_seg_kernel(LayerArgs a, SegGeom g, int S) {
    extern __shared__ __align__(128) unsigned char smem[];
    const int N = a.N;
    const int nu = a.nu;
    const int Q = N / nu;
    float* s_st = reinterpret_cast<float*>(smem);
    uint64_t* bars = reinterpret_cast<uint64_t*>(s_st + (size_t)S * g.stage);
    uint64_t* in_full = bars;
    uint64_t* out_full = bars + S;
    int* s_row = reinterpret_cast<int*>(bars + 2 * S);  // [S]
    int* s_slot = s_row + S;
    int* s_flag = s_slot + S;
    constexpr int kConsumerWarps = kSegThreads / 32;

    const int count = *a.count;
    const long long ntiles = (long long)count * g.nseg;
    const long long tpc = (ntiles + gridDim.x - 1) / gridDim.x;
    const long long t_begin = (long long)blockIdx.x * tpc;
    const int my_tiles = (int)max(0LL, min(ntiles, t_begin + tpc) - t_begin);
    if (my_tiles <= 0) return;
    if (threadIdx.x == 0) {
        for (int b = 0; b < S; ++b) {
            mbar_init(&in_full[b], 1);
            mbar_init(&out_full[b], kConsumerWarps);
        }
        fence_proxy_async_smem();
    }
    __syncthreads();

    if (threadIdx.x >= kSegThreads) {
        // ------------------------------------------------------------ producer / storer warp
        const int lane = threadIdx.x & 31;
        auto seg_range = [&](int seg, int& lo, int& n) {  // a-range (A) or residue range (C)
            if (g.cseg == 0) {
                lo = seg * g.A_T;
                n = min(g.A_T, Q - lo);
            } else {
                lo = seg * g.C_T;
                n = min(g.C_T, nu - lo);
            }
        };
        auto load = [&](int j) {
            const int b = j % S;
            const long long tile = t_begin + j;
            const int pos = (int)(tile / g.nseg), seg = (int)(tile % g.nseg);
            const int row = a.rows[pos];
            int lo, n;
            seg_range(seg, lo, n);
            const float* gr = a.yin + (size_t)row * N;
            float* st = s_st + (size_t)b * g.stage;
            uint32_t bytes;
            if (g.cseg == 0) {
                const long long f0 = (long long)lo * nu;
                const long long f1 = (long long)(lo + n + kSK) * nu;  // exclusive, may pass N (wraps)
                bytes = (uint32_t)((f1 - f0) * 4);
                if (lane == 0) {
                    s_row[b] = row;
                    s_flag[b] = 0;
                    if constexpr (MODE == MODE_RESIDUAL) s_slot[b] = a.cslot[row];
                    mbar_arrive_expect_tx(&in_full[b], bytes);
                    const long long e0 = min(f1, (long long)N);
                    bulk_g2s(st, gr + f0, (uint32_t)((e0 - f0) * 4), &in_full[b]);
                    long long done = e0 - f0;
                    while (f0 + done < f1) {  // wrap: continue from the row head
                        const long long len = min(f1 - f0 - done, (long long)N);
                        bulk_g2s(st + done, gr, (uint32_t)(len * 4), &in_full[b]);
                        done += len;
                    }
                }
            } else {
                bytes = (uint32_t)g.rows_st * (uint32_t)n * 4;
                if (lane == 0) {
                    s_row[b] = row;
                    s_flag[b] = 0;
                    if constexpr (MODE == MODE_RESIDUAL) s_slot[b] = a.cslot[row];
                    mbar_arrive_expect_tx(&in_full[b], bytes);
                }
                __syncwarp();
                for (int r = lane; r < g.rows_st; r += 32)
                    bulk_g2s(st + (size_t)r * g.P, gr + (size_t)(r % Q) * nu + lo, (uint32_t)n * 4, &in_full[b]);
            }
            __syncwarp();
        };
        auto store = [&](int j) {
            const int b = j % S;
            const long long tile = t_begin + j;
            const int pos = (int)(tile / g.nseg), seg = (int)(tile % g.nseg);
            int lo, n;
            seg_range(seg, lo, n);
            if (lane == 0) mbar_wait(&out_full[b], (uint32_t)((j / S) & 1));
            __syncwarp();
            const int row = s_row[b];
            float* gr = a.yout + (size_t)row * N;
            const float* st = s_st + (size_t)b * g.stage;
            if (g.cseg == 0) {
                if (lane == 0) bulk_s2g(gr + (size_t)lo * nu, st, (uint32_t)n * nu * 4);
            } else {
                for (int r = lane; r < Q; r += 32) bulk_s2g(gr + (size_t)r * nu + lo, st + (size_t)r * g.P, (uint32_t)n * 4);
            }
            if (lane == 0 && s_flag[b]) {
                if (a.flag_pos) a.flag_pos[pos] = 1;
                if (a.flag_row) a.flag_row[row] = 1;
            }
            bulk_commit();
            bulk_wait_read0();  // this lane's stores have read the stage
            __syncwarp();
        };
        for (int j = 0; j < my_tiles; ++j) {
            if (j >= S) store(j - S);
            load(j);
        }
        for (int j = max(0, my_tiles - S); j < my_tiles; ++j) store(j);
        bulk_wait0();
        return;
    }

    // ---------------------------------------------------------------- consumers
    float w[UNIF ? 1 : kSK];
    if constexpr (!UNIF) {
#pragma unroll
        for (int n = 0; n < kSK; ++n) w[n] = __ldg(a.wtab + n);
    }
    const float w0 = a.w0;
    const float b0 = UBIAS ? __ldg(a.bias) : 0.0f;
    const int lane = threadIdx.x & 31;
    const int item = threadIdx.x;
    const int P = g.P;
    for (int j = 0; j < my_tiles; ++j) {
        const int b = j % S;
        const long long tile = t_begin + j;
        const int seg = (int)(tile % g.nseg);
        mbar_wait(&in_full[b], (uint32_t)((j / S) & 1));
        float* st = s_st + (size_t)b * g.stage;
        const int row = s_row[b];
        const int slot = (MODE == MODE_RESIDUAL) ? s_slot[b] : 0;
        float v[32];
        int n_out = 0, ob = 0, os = 1;
        bool have = false;
        auto fin = [&](float acc, int q, int m, bool valid) {
            const float bq = UBIAS ? b0 : __ldg(a.bias + q);
            v[m] = epilogue<MODE>(a, acc, bq, q, row, slot, valid);
        };
        if (g.cls == 0) {  // nu == 1, A-segment: outputs a in [lo + 17 it, ...)
            constexpr int M = 17, WIN = M + kSK - 1;
            const int lo = seg * g.A_T, n = min(g.A_T, Q - lo);
            const int a0 = item * M;
            if (a0 < n) {
                have = true;
                float R[WIN];
#pragma unroll
                for (int i = 0; i < WIN; ++i) R[i] = st[a0 + i];
                n_out = min(M, n - a0);
                ob = a0;
                os = 1;
#pragma unroll
                for (int m = 0; m < M; ++m) {
                    float acc = 0.0f;
#pragma unroll
                    for (int k = 0; k < kSK; ++k) acc = fmaf(R[m + k], UNIF ? w0 : w[k], acc);
                    fin(acc, lo + min(a0 + m, n - 1), m, a0 + m < n);
                }
            }
        } else if (g.cls == 1) {  // Q == 32, C-segment: one residue per thread, all 32 a
            const int lo = seg * g.C_T, n = min(g.C_T, nu - lo);
            if (item < n) {
                have = true;
                float R[32];
#pragma unroll
                for (int jj = 0; jj < 32; ++jj) R[jj] = st[jj * P + item];
                n_out = 32;
                ob = item;
                os = P;
#pragma unroll
                for (int m = 0; m < 32; ++m) {
                    float acc = 0.0f;
#pragma unroll
                    for (int k = 0; k < kSK; ++k) acc = fmaf(R[(m + k) & 31], UNIF ? w0 : w[k], acc);
                    fin(acc, m * nu + lo + item, m, true);
                }
            }
        } else {  // general stride, M = 16
            constexpr int M = 16, WIN = M + kSK - 1;
            int c, a0, lo_a, lo_c, na;
            bool valid;
            if (g.cseg == 0) {
                lo_a = seg * g.A_T;
                lo_c = 0;
                na = min(g.A_T, Q - lo_a);
                c = item % nu;
                a0 = (item / nu) * M;
                valid = a0 < na;
            } else {
                lo_a = 0;
                lo_c = seg * g.C_T;
                na = Q;
                const int nc = min(g.C_T, nu - lo_c);
                c = item % g.C_T;
                a0 = (item / g.C_T) * M;
                valid = c < nc && a0 < Q;
            }
            if (valid) {
                have = true;
                float R[WIN];
#pragma unroll
                for (int i = 0; i < WIN; ++i) R[i] = st[(a0 + i) * P + c];
                n_out = min(M, na - a0);
                ob = a0 * P + c;
                os = P;
#pragma unroll
                for (int m = 0; m < M; ++m) {
                    float acc = 0.0f;
#pragma unroll
                    for (int k = 0; k < kSK; ++k) acc = fmaf(R[m + k], UNIF ? w0 : w[k], acc);
                    const int am = lo_a + min(a0 + m, na - 1);
                    fin(acc, am * nu + lo_c + c, m, a0 + m < na);
                }
            }
        }
        asm volatile("bar.sync 2, %0;" ::"n"(kSegThreads) : "memory");  // all stage reads done
        float mx = 0.0f;
        if (have) {
#pragma unroll
            for (int m = 0; m < 32; ++m)
                if (m < n_out) {
                    st[ob + m * os] = v[m];
                    mx = fmaxf(mx, fabsf(v[m]));
                }
        }
        const unsigned any = __ballot_sync(0xffffffffu, mx != 0.0f);
        if (lane == 0 && any) s_flag[b] = 1;
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) mbar_arrive(&out_full[b]);
    }
}

template <int MODE, bool UNIF, bool UBIAS>
static cudaError_t launch_seg_t(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st) {
    const SegGeom g = seg_geom(a.N, a.nu);
    int S = kSegMaxStages;
    while (S > 2 && (size_t)S * g.stage * 4 + 64 * S > 110 * 1024) --S;
    const size_t smem = (size_t)S * g.stage * 4 + 2 * S * sizeof(uint64_t) + 3 * S * sizeof(int);
    auto kern = layer_circ_seg_kernel<MODE, UNIF, UBIAS>;
    int per_sm = 1;
    cudaError_t e = blocks_per_sm((const void*)kern, kSegThreads + 32, smem, &per_sm);
    if (e != cudaSuccess) return e;
    long long tiles = (long long)max_rows * g.nseg;
    int grid = num_sms * per_sm;
    if (grid > tiles) grid = (int)tiles;
    if (grid < 1) grid = 1;
    kern<<<grid, kSegThreads + 32, smem, st>>>(a, g, S);
    return cudaGetLastError();
}

template <int MODE>
static cudaError_t launch_seg_m(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st) {
    const bool unif = a.wtab == nullptr, ub = a.uniform_bias != 0;
    if (unif && ub) return launch_seg_t<MODE, true, true>(a, max_rows, num_sms, st);
    if (unif) return launch_seg_t<MODE, true, false>(a, max_rows, num_sms, st);
    if (ub) return launch_seg_t<MODE, false, true>(a, max_rows, num_sms, st);
    return launch_seg_t<MODE, false, false>(a, max_rows, num_sms, st);
}

cudaError_t launch_layer_circ_seg(const LayerArgs& a, int mode, int max_rows, int num_sms, cudaStream_t st) {
    if (max_rows <= 0) return cudaSuccess;
    switch (mode) {
        case MODE_PLAIN: return launch_seg_m<MODE_PLAIN>(a, max_rows, num_sms, st);
        case MODE_CENTROID: return launch_seg_m<MODE_CENTROID>(a, max_rows, num_sms, st);
        default: return launch_seg_m<MODE_RESIDUAL>(a, max_rows, num_sms, st);
    }
}

}  // namespace snicit
