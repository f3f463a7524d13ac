// kernels_circ_seg.cu -- circulant layer kernel for large rows (N >= ~8K: C3 = 16384, C4 = 65536).
//
// Same arithmetic as kernels_circ.cu (the stored-order fma chain of every output, reading R12), but a
// row no longer has to fit in shared memory: the row is cut into segments of about 4K outputs.
//   A-segment (nu == 1, or a general stride whose staged window is small): outputs a in [a_s, a_e)
//     (all residues c); the window holds a-rows [a_s, a_e + 32) mod Q, i.e. the contiguous float range
//     [a_s*nu, (a_e + 32)*nu) mod N (one or two TMA bulk copies), so windows never wrap.
//   C-segment (Q == 32, or a general stride with small Q): outputs for residues c in [c_s, c_s + C_T)
//     and every a; the window holds a-rows 0 .. Q + 31 (the first 31 repeated for Q > 32 windows)
//     of C_T contiguous floats each: one bulk copy per a-row, issued by all producer lanes.
// A window element (a_local, c_local) lives at a_local * P + c_local (P = nu for A-segments, C_T for
// C-segments); outputs are written back in place and TMA-stored (one copy for A-segments, one per
// a-row for C-segments).
//
// Tiles.  PAIR (PLAIN mode): a tile is (row, segment pair {s, s + half}); both windows share the
// stage and every consumer thread runs the same work item on both, the two windows' elements sharing
// a register pair, so each FMA of the chain is one FFMA2 for two outputs (per-lane rounding identical
// to fmaf).  Otherwise a tile is (row, segment).  A row's any-non-zero flag is OR-ed into
// flag_pos[list position] (plain stores of 1; the ordered compaction that reads it also clears it).
//
// Pipeline: one producer warp (S stages) and 8 consumer warps (one work item per thread), mbarrier
// full/empty handshakes, no CTA-wide barriers (as kernels_circ.cu).
#include <cuda_runtime.h>

#include "snicit_internal.cuh"

namespace snicit {

constexpr int kSegThreads = 256;
constexpr int kSK = 32;
constexpr int kSegMaxStages = 6;

struct SegGeom {
    int cseg;      // 0: A-segment, 1: C-segment
    int cls;       // 0: nu == 1, 1: Q == 32 (whole class), 2: general
    int pair;      // 1: a tile holds two segments of one row (FFMA2)
    int nseg;      // segments per row
    int tpr;       // tiles per row (nseg, or ceil(nseg / 2) when paired)
    int A_T;       // A: a-rows of outputs per segment
    int C_T;       // C: residues per segment
    int P;         // window pitch (floats per staged a-row)
    int rows_st;   // staged a-rows per window
    int sw;        // floats per window (16-byte multiple)
};

// outputs per work item: nu == 1: 17 (odd -> conflict-free); general: 16 (8 paired); Q == 32: 32
// (16 paired) outputs of one residue class per item
__host__ __device__ constexpr int seg_M(int cls, int pair) {
    return cls == 0 ? 17 : (cls == 1 ? (pair ? 16 : 32) : (pair ? 8 : 16));
}

static SegGeom seg_geom(int N, int nu, int pair) {
    SegGeom g{};
    const int Q = N / nu;
    g.cls = nu == 1 ? 0 : (Q == 32 ? 1 : 2);
    g.pair = pair;
    const int M = seg_M(g.cls, pair);
    if (g.cls == 0) {  // A-segments of 256 items x 17 outputs
        g.cseg = 0;
        g.A_T = 256 * M;
        g.P = 1;
        g.rows_st = g.A_T + kSK;  // + 31-row halo, rounded so every copy is a 16-byte multiple
    } else if (g.cls == 2 && nu <= 256 && (size_t)(256 / nu * M + kSK) * nu <= 8192) {
        g.cseg = 0;  // general stride, A-segments: nu residues x (A_T / M) chunks = 256 items
        g.A_T = (256 / nu) * M;
        g.P = nu;
        g.rows_st = g.A_T + kSK;
    } else {
        g.cseg = 1;  // C-segments: C_T residues x (items per residue)
        const int per_c = g.cls == 1 ? 32 / M : (Q + M - 1) / M;
        g.C_T = 256 / per_c;
        if (g.C_T > nu) g.C_T = nu;
        g.C_T &= ~3;  // 16-byte rows
        if (g.C_T < 4) g.C_T = 4;
        g.P = g.C_T;
        g.rows_st = g.cls == 1 ? 32 : Q + kSK - 1;
    }
    g.nseg = g.cseg == 0 ? (Q + g.A_T - 1) / g.A_T : (nu + g.C_T - 1) / g.C_T;
    g.tpr = pair ? (g.nseg + 1) / 2 : g.nseg;
    g.sw = ((g.rows_st * g.P) + 3) & ~3;
    return g;
}

bool circ_seg_supported(int N, int K, int nu) {
    if (K != kSK || nu <= 0 || N % nu != 0 || N % 4 != 0) return false;
    if ((long long)K * nu > N) return false;
    for (int pair = 0; pair < 2; ++pair) {
        const SegGeom g = seg_geom(N, nu, pair);
        if (g.cseg == 1 && (nu % 4 != 0 || g.C_T < 4)) return false;
        if (g.cseg == 0 && g.cls == 2 && (nu % 4 != 0)) return false;
        if ((size_t)g.sw * 4 * (pair ? 2 : 1) * 2 > 200 * 1024) return false;
    }
    return true;
}

template <int MODE, bool UNIF, bool UBIAS, bool PAIR>
__global__ void __launch_bounds__(kSegThreads + 32, 2) layer_circ_seg_kernel(LayerArgs a, SegGeom g, int S) {
    constexpr int NW = PAIR ? 2 : 1;  // windows per tile
    extern __shared__ __align__(128) unsigned char smem[];
    const int N = a.N;
    const int nu = a.nu;
    const int Q = N / nu;
    const int tstage = NW * g.sw;
    float* s_st = reinterpret_cast<float*>(smem);
    uint64_t* bars = reinterpret_cast<uint64_t*>(s_st + (size_t)S * tstage);
    uint64_t* in_full = bars;
    uint64_t* out_full = bars + S;
    int* s_row = reinterpret_cast<int*>(bars + 2 * S);  // [S]
    int* s_slot = s_row + S;
    int* s_flag = s_slot + S;
    unsigned* s_cmin = reinterpret_cast<unsigned*>(s_flag + S);  // [S] constant-row mode: min / max bits
    unsigned* s_cmax = s_cmin + S;
    constexpr int kConsumerWarps = kSegThreads / 32;

    const int count = *a.count;
    const long long ntiles = (long long)count * g.tpr;
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

    // segment geometry: [lo, lo + n) a-rows (A) or residues (C); segment id >= nseg: absent (n = 0)
    auto seg_range = [&](int seg, int& lo, int& n) {
        if (seg >= g.nseg) {
            lo = 0;
            n = 0;
        } else if (g.cseg == 0) {
            lo = seg * g.A_T;
            n = min(g.A_T, Q - lo);
        } else {
            lo = seg * g.C_T;
            n = min(g.C_T, nu - lo);
        }
    };
    auto win_bytes = [&](int n) -> uint32_t {
        if (n == 0) return 0u;
        return g.cseg == 0 ? (uint32_t)((n + kSK) * nu * 4) : (uint32_t)g.rows_st * (uint32_t)n * 4;
    };

    if (threadIdx.x >= kSegThreads) {
        // ------------------------------------------------------------ producer / storer warp
        const int lane = threadIdx.x & 31;
        auto load_window = [&](const float* gr, int seg, float* st, uint64_t* bar) {
            int lo, n;
            seg_range(seg, lo, n);
            if (n == 0) return;
            if (g.cseg == 0) {
                if (lane == 0) {
                    const long long f0 = (long long)lo * nu;
                    const long long f1 = (long long)(lo + n + kSK) * nu;  // exclusive, may pass N (wraps)
                    const long long e0 = min(f1, (long long)N);
                    bulk_g2s(st, gr + f0, (uint32_t)((e0 - f0) * 4), bar);
                    long long done = e0 - f0;
                    while (f0 + done < f1) {  // wrap: continue from the row head
                        const long long len = min(f1 - f0 - done, (long long)N);
                        bulk_g2s(st + done, gr, (uint32_t)(len * 4), bar);
                        done += len;
                    }
                }
            } else {
                for (int r = lane; r < g.rows_st; r += 32)
                    bulk_g2s(st + (size_t)r * g.P, gr + (size_t)(r % Q) * nu + lo, (uint32_t)n * 4, bar);
            }
        };
        auto store_window = [&](float* gr, int seg, const float* st) {
            int lo, n;
            seg_range(seg, lo, n);
            if (n == 0) return;
            if (g.cseg == 0) {
                if (lane == 0) bulk_s2g(gr + (size_t)lo * nu, st, (uint32_t)n * nu * 4);
            } else {
                for (int r = lane; r < Q; r += 32) bulk_s2g(gr + (size_t)r * nu + lo, st + (size_t)r * g.P, (uint32_t)n * 4);
            }
        };
        auto load = [&](int j) {
            const int b = j % S;
            const long long tile = t_begin + j;
            const int pos = (int)(tile / g.tpr), tp = (int)(tile % g.tpr);
            const int row = a.rows[pos];
            const int sa = tp, sb = PAIR ? tp + g.tpr : g.nseg;
            int lo, na, nb;
            seg_range(sa, lo, na);
            seg_range(sb, lo, nb);
            const float* gr = a.yin + (size_t)row * N;
            float* st = s_st + (size_t)b * tstage;
            if (lane == 0) {
                s_row[b] = row;
                s_flag[b] = 0;
                s_cmin[b] = 0xffffffffu;
                s_cmax[b] = 0u;
                if constexpr (MODE == MODE_RESIDUAL) s_slot[b] = a.cslot[row];
                mbar_arrive_expect_tx(&in_full[b], win_bytes(na) + (PAIR ? win_bytes(nb) : 0u));
            }
            __syncwarp();
            load_window(gr, sa, st, &in_full[b]);
            if constexpr (PAIR) load_window(gr, sb, st + g.sw, &in_full[b]);
            __syncwarp();
        };
        auto store = [&](int j) {
            const int b = j % S;
            const long long tile = t_begin + j;
            const int pos = (int)(tile / g.tpr), tp = (int)(tile % g.tpr);
            if (lane == 0) mbar_wait(&out_full[b], (uint32_t)((j / S) & 1));
            __syncwarp();
            const int row = s_row[b];
            float* gr = a.yout + (size_t)row * N;
            const float* st = s_st + (size_t)b * tstage;
            store_window(gr, tp, st);
            if constexpr (PAIR) store_window(gr, tp + g.tpr, st + g.sw);
            if (lane == 0 && s_flag[b]) {
                if (a.flag_pos) a.flag_pos[pos] = 1;
                if (a.flag_row) a.flag_row[row] = 1;
            }
            if (lane == 0 && a.cmin) {  // constant-row mode: this tile's (min, max) into the row's
                atomicMin(a.cmin + pos, s_cmin[b]);
                atomicMax(a.cmax + pos, s_cmax[b]);
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
    constexpr int MG = seg_M(2, PAIR);  // general class
    constexpr int OQ = seg_M(1, PAIR);  // Q == 32 class
    constexpr int VM = 32;              // max outputs per item
    float w[UNIF ? 1 : kSK];
    if constexpr (!UNIF) {
#pragma unroll
        for (int n = 0; n < kSK; ++n) w[n] = __ldg(a.wtab + n);
    }
    const float w0 = a.w0;
    const float b0 = UBIAS ? __ldg(a.bias) : 0.0f;
    const unsigned long long W2 = f2_pack(w0, w0);
    const int lane = threadIdx.x & 31;
    const int item = threadIdx.x;
    const int P = g.P;
    for (int j = 0; j < my_tiles; ++j) {
        const int b = j % S;
        const long long tile = t_begin + j;
        const int tp = (int)(tile % g.tpr);
        mbar_wait(&in_full[b], (uint32_t)((j / S) & 1));
        float* stA = s_st + (size_t)b * tstage;
        float* stB = stA + g.sw;  // PAIR only
        const int row = s_row[b];
        const int slot = (MODE == MODE_RESIDUAL) ? s_slot[b] : 0;
        int loA, nA, loB = 0, nB = 0;
        seg_range(tp, loA, nA);
        if constexpr (PAIR) seg_range(tp + g.tpr, loB, nB);
        float v0[VM], v1[PAIR ? VM : 1];
        int nv0 = 0, nv1 = 0, ob = 0, os = 1;
        // one output of the single window: global index q, validity (no side effects if invalid)
        auto fin1 = [&](float acc, int q, int m, bool valid) {
            const float bq = UBIAS ? b0 : __ldg(a.bias + q);
            v0[m] = epilogue<MODE>(a, acc, bq, q, row, slot, valid);
        };
        // one output of each of the two windows (PLAIN only): FADD2 + clamp
        auto fin2 = [&](unsigned long long acc, int qa, int qb, int m) {
            float z0, z1;
            const float ba = UBIAS ? b0 : __ldg(a.bias + qa), bb = UBIAS ? b0 : __ldg(a.bias + qb);
            f2_unpack(f2_add(acc, f2_pack(ba, bb)), z0, z1);
            v0[m] = sigma(z0, a.ymax);
            if constexpr (PAIR) v1[m] = sigma(z1, a.ymax);
        };
        if (g.cls == 0) {  // nu == 1, A-segment: outputs a in [lo + 17 item, ...)
            constexpr int M = 17, WIN = M + kSK - 1;
            const int a0 = item * M;
            if (a0 < max(nA, nB)) {
                nv0 = max(0, min(M, nA - a0));
                nv1 = max(0, min(M, nB - a0));
                ob = a0;
                os = 1;
                if constexpr (PAIR) {
                    unsigned long long R[WIN];
#pragma unroll
                    for (int i = 0; i < WIN; ++i) R[i] = f2_pack(stA[a0 + i], stB[a0 + i]);
#pragma unroll
                    for (int m = 0; m < M; ++m) {
                        unsigned long long acc = 0ull;
#pragma unroll
                        for (int k = 0; k < kSK; ++k) acc = f2_fma(R[m + k], W2, acc);
                        fin2(acc, loA + min(a0 + m, max(nA, 1) - 1), loB + min(a0 + m, max(nB, 1) - 1), m);
                    }
                } else {
                    float R[WIN];
#pragma unroll
                    for (int i = 0; i < WIN; ++i) R[i] = stA[a0 + i];
#pragma unroll
                    for (int m = 0; m < M; ++m) {
                        float acc = 0.0f;
#pragma unroll
                        for (int k = 0; k < kSK; ++k) acc = fmaf(R[m + k], UNIF ? w0 : w[k], acc);
                        fin1(acc, loA + min(a0 + m, nA - 1), m, a0 + m < nA);
                    }
                }
            }
        } else if (g.cls == 1) {  // Q == 32, C-segment: OQ outputs of one residue class per item
            const int cc = item % g.C_T, g0 = (item / g.C_T) * OQ;
            if (g0 < 32 && cc < max(nA, nB)) {
                nv0 = cc < nA ? OQ : 0;
                nv1 = cc < nB ? OQ : 0;
                ob = g0 * P + cc;
                os = P;
                if constexpr (PAIR) {
                    unsigned long long R[32];
#pragma unroll
                    for (int jj = 0; jj < 32; ++jj) {
                        const int ro = ((g0 + jj) & 31) * P + cc;  // rotated: compile-time indices below
                        R[jj] = f2_pack(stA[ro], stB[ro]);
                    }
#pragma unroll
                    for (int m = 0; m < OQ; ++m) {
                        unsigned long long acc = 0ull;
#pragma unroll
                        for (int k = 0; k < kSK; ++k) acc = f2_fma(R[(m + k) & 31], W2, acc);
                        fin2(acc, (g0 + m) * nu + loA + min(cc, max(nA, 1) - 1),
                             (g0 + m) * nu + loB + min(cc, max(nB, 1) - 1), m);
                    }
                } else {
                    float R[32];
#pragma unroll
                    for (int jj = 0; jj < 32; ++jj) R[jj] = stA[((g0 + jj) & 31) * P + cc];
#pragma unroll
                    for (int m = 0; m < OQ; ++m) {
                        float acc = 0.0f;
#pragma unroll
                        for (int k = 0; k < kSK; ++k) acc = fmaf(R[(m + k) & 31], UNIF ? w0 : w[k], acc);
                        fin1(acc, (g0 + m) * nu + loA + min(cc, nA - 1), m, cc < nA);
                    }
                }
            }
        } else {  // general stride
            constexpr int M = MG, WIN = M + kSK - 1;
            int c, a0;
            bool active;
            if (g.cseg == 0) {
                c = item % nu;
                a0 = (item / nu) * M;
                active = a0 < max(nA, nB);
                nv0 = max(0, min(M, nA - a0));
                nv1 = max(0, min(M, nB - a0));
            } else {
                c = item % g.C_T;
                a0 = (item / g.C_T) * M;
                active = a0 < Q && c < max(nA, nB);
                nv0 = c < nA ? min(M, Q - a0) : 0;
                nv1 = c < nB ? min(M, Q - a0) : 0;
            }
            if (active) {
                ob = a0 * P + c;
                os = P;
                // global index of output m of a window (segment lo, n), clamped for discarded outputs
                auto gq = [&](int lo, int n, int m) -> int {
                    if (g.cseg == 0) return (lo + min(a0 + m, max(n, 1) - 1)) * nu + c;
                    return min(a0 + m, Q - 1) * nu + lo + min(c, max(n, 1) - 1);
                };
                if constexpr (PAIR) {
                    unsigned long long R[WIN];
#pragma unroll
                    for (int i = 0; i < WIN; ++i) R[i] = f2_pack(stA[(a0 + i) * P + c], stB[(a0 + i) * P + c]);
#pragma unroll
                    for (int m = 0; m < M; ++m) {
                        unsigned long long acc = 0ull;
#pragma unroll
                        for (int k = 0; k < kSK; ++k) acc = f2_fma(R[m + k], W2, acc);
                        fin2(acc, gq(loA, nA, m), gq(loB, nB, m), m);
                    }
                } else {
                    float R[WIN];
#pragma unroll
                    for (int i = 0; i < WIN; ++i) R[i] = stA[(a0 + i) * P + c];
#pragma unroll
                    for (int m = 0; m < M; ++m) {
                        float acc = 0.0f;
#pragma unroll
                        for (int k = 0; k < kSK; ++k) acc = fmaf(R[m + k], UNIF ? w0 : w[k], acc);
                        fin1(acc, gq(loA, nA, m), m, m < nv0);
                    }
                }
            } else {
                nv0 = nv1 = 0;
            }
        }
        asm volatile("bar.sync 2, %0;" ::"n"(kSegThreads) : "memory");  // all stage reads done
        float mx = 0.0f, mn = a.ymax;
        if (PAIR && g.cls == 0) {
            // nu == 1, two windows: unguarded stores (outputs past a window's segment land in the
            // window's halo, an absent second window's buffer is never stored); max of the valid ones
            constexpr int M = 17;
            if (nv0 > 0 || nv1 > 0) {
#pragma unroll
                for (int m = 0; m < M; ++m) {
                    stA[ob + m] = v0[m];
                    stB[ob + m] = v1[PAIR ? m : 0];
                }
                if (nv0 == M && nv1 == M) {
#pragma unroll
                    for (int m = 0; m < M; ++m) mx = fmaxf(mx, fmaxf(v0[m], v1[PAIR ? m : 0]));
                    if (a.cmin) {
#pragma unroll
                        for (int m = 0; m < M; ++m) mn = fminf(mn, fminf(v0[m], v1[PAIR ? m : 0]));
                    }
                } else {
#pragma unroll
                    for (int m = 0; m < M; ++m) {
                        if (m < nv0) {
                            mx = fmaxf(mx, fabsf(v0[m]));
                            mn = fminf(mn, v0[m]);
                        }
                        if (m < nv1) {
                            mx = fmaxf(mx, fabsf(v1[PAIR ? m : 0]));
                            mn = fminf(mn, v1[PAIR ? m : 0]);
                        }
                    }
                }
            }
        } else {
#pragma unroll
            for (int m = 0; m < VM; ++m) {
                if (m < nv0) {
                    stA[ob + m * os] = v0[m];
                    mx = fmaxf(mx, fabsf(v0[m]));
                    mn = fminf(mn, v0[m]);
                }
                if constexpr (PAIR) {
                    if (m < nv1) {
                        stB[ob + m * os] = v1[m];
                        mx = fmaxf(mx, fabsf(v1[m]));
                        mn = fminf(mn, v1[m]);
                    }
                }
            }
        }
        const unsigned any = __ballot_sync(0xffffffffu, mx != 0.0f);
        if (lane == 0 && any) s_flag[b] = 1;
        if (MODE == MODE_PLAIN && a.cmin) {  // constant-row mode: the tile's output range (bits, -0 -> +0)
#pragma unroll
            for (int d = 16; d; d >>= 1) {
                mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, d));
                mn = fminf(mn, __shfl_xor_sync(0xffffffffu, mn, d));
            }
            if (lane == 0) {
                atomicMin(&s_cmin[b], __float_as_uint(mn + 0.0f));
                atomicMax(&s_cmax[b], __float_as_uint(mx + 0.0f));
            }
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) mbar_arrive(&out_full[b]);
    }
}

template <int MODE, bool UNIF, bool UBIAS, bool PAIR>
static cudaError_t launch_seg_t(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st) {
    const SegGeom g = seg_geom(a.N, a.nu, PAIR ? 1 : 0);
    const size_t tstage = (size_t)(PAIR ? 2 : 1) * g.sw * 4;
    int S = kSegMaxStages;
    while (S > 2 && (size_t)S * tstage + 64 * S > 110 * 1024) --S;
    const size_t smem = (size_t)S * tstage + 2 * S * sizeof(uint64_t) + 5 * S * sizeof(int);
    auto kern = layer_circ_seg_kernel<MODE, UNIF, UBIAS, PAIR>;
    int per_sm = 1;
    cudaError_t e = blocks_per_sm((const void*)kern, kSegThreads + 32, smem, &per_sm);
    if (e != cudaSuccess) return e;
    long long tiles = (long long)max_rows * g.tpr;
    int grid = num_sms * per_sm;
    if (grid > tiles) grid = (int)tiles;
    if (grid < 1) grid = 1;
    kern<<<grid, kSegThreads + 32, smem, st>>>(a, g, S);
    return cudaGetLastError();
}

template <int MODE>
static cudaError_t launch_seg_m(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st) {
    const bool unif = a.wtab == nullptr, ub = a.uniform_bias != 0;
    // paired segments (FFMA2) for nu == 1 PLAIN layers: measured faster there; for the strided classes
    // the paired windows halve the copy granularity and the kernel becomes copy-issue-bound
    const bool pair = MODE == MODE_PLAIN && unif && a.nu == 1;
    if (pair && ub) return launch_seg_t<MODE, true, true, MODE == MODE_PLAIN>(a, max_rows, num_sms, st);
    if (pair) return launch_seg_t<MODE, true, false, MODE == MODE_PLAIN>(a, max_rows, num_sms, st);
    if (unif && ub) return launch_seg_t<MODE, true, true, false>(a, max_rows, num_sms, st);
    if (unif) return launch_seg_t<MODE, true, false, false>(a, max_rows, num_sms, st);
    if (ub) return launch_seg_t<MODE, false, true, false>(a, max_rows, num_sms, st);
    return launch_seg_t<MODE, false, false, false>(a, max_rows, num_sms, st);
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
