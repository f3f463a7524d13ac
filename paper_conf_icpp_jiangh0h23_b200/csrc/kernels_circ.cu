// kernels_circ.cu -- the fused layer kernel for shift-invariant (circulant) layers, sm_100a.
//
// A layer is circulant when output column j reads inputs (j + n*nu) mod N, n = 0..K-1 (K = 32),
// with per-n weights -- the RadiX-Net-like SDGC layers "sums of cyclic permutations".
// Writing j = a*nu + c (Q = N/nu), output (a, c) reads (a + n mod Q, c): every residue class c is
// an independent circular sliding window of length K over Q values.  A thread loads a window of
// WIN inputs of one class into registers and produces M outputs from it, so each staged input
// element is read from shared memory WIN/M times instead of K times, and the FMA chain of every
// output is evaluated exactly in the stored order n = 0..K-1 (R12: acc = fmaf(y, w_n, acc)).
//
// Stride classes (template CLS):
//   NU1  nu == 1: lanes walk chunk starts 17 apart (odd -> conflict-free LDS); the staged row gets a
//        64-float circular halo (a second TMA copy of the row head) so windows never wrap.
//   Q32  Q == 32: one thread owns a whole residue class (32 loads, 32 outputs, all rotations at
//        compile time); lanes walk consecutive residues.
//   GEN  other nu: M = 16 outputs per thread, lanes walk consecutive residues; windows that wrap
//        (warp-uniform) take a masked path.
//
// Pipeline per CTA (persistent over a contiguous range of row tiles, warp-specialised): a producer
// warp keeps S - 1 tiles of TMA bulk loads in flight while 8 consumer warps compute; the outputs
// overwrite the tile's stage in shared memory and the producer writes them back with TMA bulk stores
// (coalesced for every nu).  Producer and consumers synchronise only through mbarriers.
#include <cuda_runtime.h>

#include "snicit_internal.cuh"

namespace snicit {

constexpr int kCircThreads = 256;
constexpr int kK = 32;      // taps per column (SDGC: 32 connections per neuron)
constexpr int kHalo = 64;   // floats appended to each staged row for NU1 (>= M + K - 2 = 47)

enum CircClass : int { CLS_NU1 = 0, CLS_Q32 = 1, CLS_GEN = 2 };
template <int CLS>
struct CircCfg;
template <>
struct CircCfg<CLS_NU1> {
    static constexpr int M = 17, WIN = M + kK - 1;
};
template <>
struct CircCfg<CLS_Q32> {
    static constexpr int M = 32, WIN = 32;
};
template <>
struct CircCfg<CLS_GEN> {
    static constexpr int M = 16, WIN = M + kK - 1;
};

// Circular halo appended to each staged row (a second TMA copy of the row head) so sliding windows
// never wrap: nu == 1 -> 64 floats; general class -> WIN - 1 = 46 whole a-rows (46 * nu floats) when
// that is at most the row itself (Q >= 46); Q == 32 class -> none (rotations are compile-time).
__host__ __device__ constexpr int circ_halo(int N, int cls, int nu) {
    return cls == CLS_NU1 ? kHalo : (cls == CLS_GEN && 46 * nu <= N && nu % 2 == 0 ? 46 * nu : 0);
}
__host__ __device__ constexpr int circ_stride(int N, int cls, int nu) { return N + circ_halo(N, cls, nu); }

constexpr int kMaxStages = 8;
constexpr int kSurvCap = 256;  // per-CTA buffer of surviving row ids (fused dead-row compaction)
// Shared-memory layout (per CTA): stage[S][RT][stride] | mbarriers (2S) | row/slot/flag [S][RT] | surv[256]
__host__ __device__ constexpr size_t circ_smem2(int N, int cls, int nu, int RT, int S) {
    return sizeof(float) * (size_t)S * RT * circ_stride(N, cls, nu) + 2 * (size_t)S * sizeof(uint64_t) +
           3 * (size_t)S * sizeof(int) * (size_t)RT + sizeof(int) * kSurvCap;
}

__device__ __forceinline__ void consumer_bar() { asm volatile("bar.sync 1, %0;" ::"n"(kCircThreads) : "memory"); }

// Warp-aggregated row flags: lane 0 sets flag[r] for every row r that some lane reported non-zero, so
// the only writer of a flag is the lane that then arrives on the mbarrier (release) -- the producer's
// acquire sees it without relying on cross-lane ordering.  `nz`/`r` per lane; warp-uniform loop.
__device__ __forceinline__ void warp_flag_rows(int* flags, bool nz, int r) {
    unsigned m = __ballot_sync(0xffffffffu, nz);
    while (m) {
        const int src = __ffs(m) - 1;
        const int rs = __shfl_sync(0xffffffffu, r, src);
        m &= ~__ballot_sync(0xffffffffu, r == rs);
        if ((threadIdx.x & 31) == 0) flags[rs] = 1;
    }
}

// Warp-specialised, in-place: warps 0..7 compute (one work item per thread per tile), warp 8 is the
// producer/storer.  Tile j of this CTA lives in stage j % S (k-th use: parity k & 1):
//   in_full[s]   producer arrive.expect_tx + TMA load bytes  -> consumers may read stage s
//   out_full[s]  one arrive per consumer warp (after the outputs were written into stage s and
//                proxy-fenced)                                -> producer TMA-stores stage s; once the
//                store has read it (bulk wait_group.read) the producer reloads the stage.
// Consumers keep their M outputs in registers, meet at a consumer-only named barrier (every read of
// the stage is done), then overwrite the stage with the outputs, so no separate output buffers are
// needed and more stages (bytes in flight) fit.  The producer keeps S - 1 tiles of loads ahead.
// PAIR (PLAIN mode): each consumer thread runs its work item on two rows of the tile at once, the
// two rows' window elements sharing a register pair, so every FMA of the chain is one FFMA2 issue
// for two outputs (per-lane rounding identical to fmaf).
template <int MODE, int CLS, bool UNIF, bool UBIAS, int NUCT, bool PAIR>
__global__ void __launch_bounds__(kCircThreads + 32, (MODE == MODE_PLAIN && UNIF) ? 3 : 2)
    layer_circ_kernel(LayerArgs a, int RT, int S) {
    constexpr int M = CircCfg<CLS>::M;
    constexpr int WIN = CircCfg<CLS>::WIN;
    extern __shared__ __align__(128) unsigned char smem[];
    const int N = a.N;
    const int nu = NUCT ? NUCT : a.nu;
    const int Q = N / nu;
    const int halo = circ_halo(N, CLS, nu);
    const int stride = N + halo;
    float* s_st = reinterpret_cast<float*>(smem);
    uint64_t* bars = reinterpret_cast<uint64_t*>(s_st + (size_t)S * RT * stride);
    uint64_t* in_full = bars;
    uint64_t* out_full = bars + S;
    int* s_row = reinterpret_cast<int*>(bars + 2 * S);
    int* s_slot = s_row + S * RT;
    int* s_flag = s_slot + S * RT;
    int* s_surv = s_flag + S * RT;
    constexpr int kConsumerWarps = kCircThreads / 32;

    const int chunks = (CLS == CLS_Q32) ? 1 : (Q + M - 1) / M;
    const int ipr = nu * chunks;  // work items per row (RT / (1 + PAIR) * ipr <= kCircThreads by the plan)
    constexpr int RPI = PAIR ? 2 : 1;  // rows per work item
    const int count = *a.count;
    const int ntiles = (count + RT - 1) / RT;
    // contiguous tile range per CTA: its row ids are contiguous in the list (prefetchable)
    const int tpc = (ntiles + (int)gridDim.x - 1) / (int)gridDim.x;
    const int t_begin = (int)blockIdx.x * tpc;
    const int my_tiles = min(ntiles, t_begin + tpc) - t_begin;
    if (my_tiles <= 0) return;

    if (threadIdx.x == 0) {
        for (int b = 0; b < S; ++b) {
            mbar_init(&in_full[b], 1);
            mbar_init(&out_full[b], kConsumerWarps);
        }
        fence_proxy_async_smem();
    }
    __syncthreads();

    if (threadIdx.x >= kCircThreads) {
        // ------------------------------------------------------------ producer / storer warp
        const int lane = threadIdx.x & 31;
        if (blockIdx.x == 0 && lane == 0 && a.zero_count) *a.zero_count = 0;  // next layer's append counter
        int nsurv = 0;  // lane 0: surviving rows buffered in s_surv
        const int row_base = t_begin * RT;  // first list position of this CTA
        const int my_rows = min(count, (t_begin + my_tiles) * RT) - row_base;
        // register windows of row ids (and centroid slots): lane l holds local position w0 + l (cur)
        // and w0 + 32 + l (nxt); the global loads of a window are issued 32 positions ahead of use
        int w0 = 0;
        int cur = lane < my_rows ? a.rows[row_base + lane] : 0;
        int nxt = 32 + lane < my_rows ? a.rows[row_base + 32 + lane] : 0;
        int scur = 0;
        if constexpr (MODE == MODE_RESIDUAL) scur = lane < my_rows ? a.cslot[cur] : 0;
        auto advance_to = [&](int p) {  // warp-uniform, p non-decreasing
            while (p >= w0 + 32) {
                cur = nxt;
                w0 += 32;
                nxt = (w0 + 32 + lane < my_rows) ? a.rows[row_base + w0 + 32 + lane] : 0;
                if constexpr (MODE == MODE_RESIDUAL) scur = (w0 + lane < my_rows) ? a.cslot[cur] : 0;
            }
        };
        auto load = [&](int j) {  // stage j % S is free (its previous tile was stored and read)
            const int b = j % S;
            const int r0 = (t_begin + j) * RT;
            const int nr = min(RT, count - r0);
            const uint32_t bytes = (uint32_t)nr * (uint32_t)((N + halo) * 4);
            if (lane == 0) mbar_arrive_expect_tx(&in_full[b], bytes);
            for (int i = 0; i < nr; ++i) {
                const int p = r0 + i - row_base;
                advance_to(p);
                const int row = __shfl_sync(0xffffffffu, cur, p - w0);
                int slot = 0;
                if constexpr (MODE == MODE_RESIDUAL) slot = __shfl_sync(0xffffffffu, scur, p - w0);
                if (lane == 0) {
                    s_row[b * RT + i] = row;
                    s_flag[b * RT + i] = 0;
                    if constexpr (MODE == MODE_RESIDUAL) s_slot[b * RT + i] = slot;
                    const float* g = a.yin + (size_t)row * N;
                    float* d = s_st + (size_t)(b * RT + i) * stride;
                    bulk_g2s(d, g, N * 4, &in_full[b]);
                    if (halo) bulk_g2s(d + N, g, halo * 4, &in_full[b]);  // circular halo
                }
            }
        };
        auto store = [&](int j) {
            if (lane == 0) {
                const int b = j % S;
                const int r0 = (t_begin + j) * RT;
                const int nr = min(RT, count - r0);
                mbar_wait(&out_full[b], (uint32_t)((j / S) & 1));
                for (int i = 0; i < nr; ++i) {
                    const int row = s_row[b * RT + i];
                    bulk_s2g(a.yout + (size_t)row * N, s_st + (size_t)(b * RT + i) * stride, N * 4);
                    const uint8_t f = s_flag[b * RT + i] ? 1 : 0;
                    if (a.flag_pos) a.flag_pos[r0 + i] = f;
                    if (a.flag_row) a.flag_row[row] = f;
                    if (a.app_list && f) s_surv[nsurv++] = row;
                }
                bulk_commit();
                bulk_wait_read0();  // the TMA engine has read the stage: it may be reloaded
            }
            __syncwarp();
        };
        // append the buffered survivors to the next active list: one atomic per batch (warp-wide copy)
        auto flush = [&](bool force) {
            const int n = __shfl_sync(0xffffffffu, nsurv, 0);
            if (n == 0 || (!force && n <= kSurvCap - RT)) return;
            int pos = 0;
            if (lane == 0) pos = atomicAdd(a.app_count, n);
            pos = __shfl_sync(0xffffffffu, pos, 0);
            for (int i = lane; i < n; i += 32) a.app_list[pos + i] = s_surv[i];
            __syncwarp();
            nsurv = 0;
        };
        for (int j = 0; j < my_tiles; ++j) {
            if (j >= S) {
                store(j - S);
                if (a.app_list) flush(false);
            }
            load(j);
        }
        for (int j = max(0, my_tiles - S); j < my_tiles; ++j) {
            store(j);
            if (a.app_list) flush(false);
        }
        if (a.app_list) flush(true);
        if (lane == 0) bulk_wait0();
        return;
    }

    // ---------------------------------------------------------------- consumers (compute)
    float w[UNIF ? 1 : kK];
    if constexpr (!UNIF) {
#pragma unroll
        for (int n = 0; n < kK; ++n) w[n] = __ldg(a.wtab + n);
    }
    const float w0 = a.w0;
    const float b0 = UBIAS ? __ldg(a.bias) : 0.0f;
    const int lane = threadIdx.x & 31;
    const int item = threadIdx.x;
    for (int j = 0; j < my_tiles; ++j) {
        const int sb = j % S;
        const int nr = min(RT, count - (t_begin + j) * RT);
        mbar_wait(&in_full[sb], (uint32_t)((j / S) & 1));
        float* st = s_st + (size_t)sb * RT * stride;
        const int n_items = ((nr + RPI - 1) / RPI) * ipr;
        if constexpr (PAIR) {
            // ---------------- two rows per item (rows rr, rr + 1 of the tile), FFMA2 chains
            float v0[M], v1[M];
            int rr = 0, obase = 0, ostep = 1, mlim = 0;
            if (item < n_items) {
                rr = (item / ipr) * 2;
                const int rem = item - (item / ipr) * ipr;
                const float* r0 = st + (size_t)rr * stride;
                const float* r1 = r0 + stride;  // rr + 1 may be past nr: in-bounds garbage, never stored
                const unsigned long long W2 = f2_pack(w0, w0);
                auto finish = [&](unsigned long long acc, int q, float& o0, float& o1) {
                    const float bq = UBIAS ? b0 : __ldg(a.bias + q);
                    float z0, z1;
                    f2_unpack(f2_add(acc, f2_pack(bq, bq)), z0, z1);
                    o0 = sigma(z0, a.ymax);
                    o1 = sigma(z1, a.ymax);
                };
                if constexpr (CLS == CLS_NU1) {
                    const int a0 = rem * M;
                    unsigned long long R[WIN];
#pragma unroll
                    for (int i = 0; i < WIN; ++i) R[i] = f2_pack(r0[a0 + i], r1[a0 + i]);
                    obase = a0;
                    ostep = 1;
                    mlim = min(M, N - a0);
#pragma unroll
                    for (int m = 0; m < M; ++m) {
                        unsigned long long acc = 0ull;
#pragma unroll
                        for (int n = 0; n < kK; ++n) acc = f2_fma(R[m + n], UNIF ? W2 : f2_pack(w[n], w[n]), acc);
                        finish(acc, min(a0 + m, N - 1), v0[m], v1[m]);
                    }
                } else if constexpr (CLS == CLS_Q32) {
                    const int c = rem;
                    unsigned long long R[32];
#pragma unroll
                    for (int jj = 0; jj < 32; ++jj) R[jj] = f2_pack(r0[jj * nu + c], r1[jj * nu + c]);
                    obase = c;
                    ostep = nu;
                    mlim = 32;
#pragma unroll
                    for (int m = 0; m < 32; ++m) {
                        unsigned long long acc = 0ull;
#pragma unroll
                        for (int n = 0; n < kK; ++n)
                            acc = f2_fma(R[(m + n) & 31], UNIF ? W2 : f2_pack(w[n], w[n]), acc);
                        finish(acc, m * nu + c, v0[m], v1[m]);
                    }
                } else {  // CLS_GEN
                    const int c = rem % nu;
                    const int a0 = (rem / nu) * M;
                    unsigned long long R[WIN];
                    if (halo || a0 + WIN <= Q) {
#pragma unroll
                        for (int i = 0; i < WIN; ++i) R[i] = f2_pack(r0[(a0 + i) * nu + c], r1[(a0 + i) * nu + c]);
                    } else {
#pragma unroll
                        for (int i = 0; i < WIN; ++i) {
                            int ai = a0 + i;
                            ai = ai >= Q ? ai - Q : ai;
                            ai = ai >= Q ? ai - Q : ai;
                            R[i] = f2_pack(r0[ai * nu + c], r1[ai * nu + c]);
                        }
                    }
                    obase = a0 * nu + c;
                    ostep = nu;
                    mlim = min(M, Q - a0);
#pragma unroll
                    for (int m = 0; m < M; ++m) {
                        unsigned long long acc = 0ull;
#pragma unroll
                        for (int n = 0; n < kK; ++n) acc = f2_fma(R[m + n], UNIF ? W2 : f2_pack(w[n], w[n]), acc);
                        finish(acc, min(a0 + m, Q - 1) * nu + c, v0[m], v1[m]);
                    }
                }
            }
            consumer_bar();  // every read of this stage is done: overwrite it with the outputs
            float mx0 = 0.0f, mx1 = 0.0f;
            const bool second = rr + 1 < nr;
            if (item < n_items) {
                static_assert(CLS == CLS_NU1, "PAIR: nu == 1 (ostep 1, outputs a0 .. a0 + M - 1)");
                // unguarded stores: tail outputs (m >= mlim) land in the row's halo and the second row
                // of an odd tail in the tile's unused row slot -- neither is ever TMA-stored
                float* d0 = st + (size_t)rr * stride + obase;
                float* d1 = d0 + stride;
#pragma unroll
                for (int m = 0; m < M; ++m) {
                    d0[m] = v0[m];
                    d1[m] = v1[m];
                }
                if (mlim == M) {  // outputs are >= 0 (sigma), so max == max |.|
#pragma unroll
                    for (int m = 0; m < M; ++m) {
                        mx0 = fmaxf(mx0, v0[m]);
                        mx1 = fmaxf(mx1, v1[m]);
                    }
                } else {
#pragma unroll
                    for (int m = 0; m < M; ++m)
                        if (m < mlim) {
                            mx0 = fmaxf(mx0, v0[m]);
                            mx1 = fmaxf(mx1, v1[m]);
                        }
                }
                if (!second) mx1 = 0.0f;
            }
            warp_flag_rows(s_flag + sb * RT, mx0 != 0.0f, rr);
            warp_flag_rows(s_flag + sb * RT, second && mx1 != 0.0f, rr + 1);
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) mbar_arrive(&out_full[sb]);
            continue;
        }
        float v[M];
        int rr = 0, obase = 0, ostep = 1, mlim = 0;
        float mx = 0.0f;
        if (item < nr * ipr) {
            rr = item / ipr;
            const int rem = item - rr * ipr;
            const int row = s_row[sb * RT + rr];
            const int slot = (MODE == MODE_RESIDUAL) ? s_slot[sb * RT + rr] : 0;
            const float* src0 = st + (size_t)rr * stride;
            if constexpr (CLS == CLS_NU1) {
                const int a0 = rem * M;
                const float* src = src0 + a0;
                float R[WIN];
#pragma unroll
                for (int i = 0; i < WIN; ++i) R[i] = src[i];
                obase = a0;
                ostep = 1;
                mlim = min(M, N - a0);
#pragma unroll
                for (int m = 0; m < M; ++m) {
                    float acc = 0.0f;
#pragma unroll
                    for (int n = 0; n < kK; ++n) acc = fmaf(R[m + n], UNIF ? w0 : w[n], acc);
                    const int q = min(a0 + m, N - 1);  // tail outputs (m >= mlim) are discarded
                    const float bq = UBIAS ? b0 : __ldg(a.bias + q);
                    v[m] = epilogue<MODE>(a, acc, bq, q, row, slot, a0 + m < N);
                }
            } else if constexpr (CLS == CLS_Q32) {
                const int c = rem;
                const float* src = src0 + c;
                float R[32];
#pragma unroll
                for (int jj = 0; jj < 32; ++jj) R[jj] = src[jj * nu];
                obase = c;
                ostep = nu;
                mlim = 32;
#pragma unroll
                for (int m = 0; m < 32; ++m) {
                    float acc = 0.0f;
#pragma unroll
                    for (int n = 0; n < kK; ++n) acc = fmaf(R[(m + n) & 31], UNIF ? w0 : w[n], acc);
                    const int q = m * nu + c;
                    const float bq = UBIAS ? b0 : __ldg(a.bias + q);
                    v[m] = epilogue<MODE>(a, acc, bq, q, row, slot);
                }
            } else {  // CLS_GEN
                const int c = rem % nu;
                const int a0 = (rem / nu) * M;
                const float* src = src0 + c;
                float R[WIN];
                if (halo || a0 + WIN <= Q) {  // halo staged, or no wrap (warp-uniform: lanes share a0)
#pragma unroll
                    for (int i = 0; i < WIN; ++i) R[i] = src[(a0 + i) * nu];
                } else {
#pragma unroll
                    for (int i = 0; i < WIN; ++i) {
                        int ai = a0 + i;  // < 3Q since Q >= K and M < K
                        ai = ai >= Q ? ai - Q : ai;
                        ai = ai >= Q ? ai - Q : ai;
                        R[i] = src[ai * nu];
                    }
                }
                obase = a0 * nu + c;
                ostep = nu;
                mlim = min(M, Q - a0);
#pragma unroll
                for (int m = 0; m < M; ++m) {
                    float acc = 0.0f;
#pragma unroll
                    for (int n = 0; n < kK; ++n) acc = fmaf(R[m + n], UNIF ? w0 : w[n], acc);
                    const int q = min(a0 + m, Q - 1) * nu + c;  // tail outputs are discarded
                    const float bq = UBIAS ? b0 : __ldg(a.bias + q);
                    v[m] = epilogue<MODE>(a, acc, bq, q, row, slot, a0 + m < Q);
                }
            }
        }
        consumer_bar();  // every read of this stage is done: overwrite it with the outputs
        if (item < nr * ipr) {
            float* dst = st + (size_t)rr * stride + obase;
            if (mlim == M) {
#pragma unroll
                for (int m = 0; m < M; ++m) {
                    dst[m * ostep] = v[m];
                    mx = fmaxf(mx, fabsf(v[m]));
                }
            } else {
#pragma unroll
                for (int m = 0; m < M; ++m)
                    if (m < mlim) {
                        dst[m * ostep] = v[m];
                        mx = fmaxf(mx, fabsf(v[m]));
                    }
            }
        }
        warp_flag_rows(s_flag + sb * RT, mx != 0.0f, rr);
        fence_proxy_async_smem();  // this thread's writes -> visible to the TMA engine
        __syncwarp();
        if (lane == 0) mbar_arrive(&out_full[sb]);
    }
}

static int circ_class(int N, int nu) {
    if (nu == 1) return CLS_NU1;
    if (N / nu == 32) return CLS_Q32;
    return CLS_GEN;
}
int circ_class_of(int N, int nu) { return circ_class(N, nu); }

bool circ_supported(int N, int K, int nu) {
    if (K != kK || nu <= 0 || N % nu != 0 || N % 4 != 0) return false;
    if ((long long)K * nu > N) return false;  // distinct inputs -> Q >= K
    const int cls = circ_class(N, nu);
    if (cls == CLS_NU1 && N < kHalo) return false;
    const int Q = N / nu;
    const int M = cls == CLS_NU1 ? CircCfg<CLS_NU1>::M : (cls == CLS_Q32 ? 32 : CircCfg<CLS_GEN>::M);
    const int ipr = nu * (cls == CLS_Q32 ? 1 : (Q + M - 1) / M);
    if (ipr > kCircThreads) return false;  // one item per consumer thread (larger N: the ELL kernel)
    return circ_smem2(N, cls, nu, 1, 2) <= 220 * 1024;
}

struct CircPlan {
    int RT, S;
    size_t smem;
};

static CircPlan circ_plan(int N, int nu, bool pair) {
    const int cls = circ_class(N, nu);
    const int Q = N / nu;
    const int M = cls == CLS_NU1 ? CircCfg<CLS_NU1>::M : (cls == CLS_Q32 ? 32 : CircCfg<CLS_GEN>::M);
    const int ipr = nu * (cls == CLS_Q32 ? 1 : (Q + M - 1) / M);
    const int rpi = pair ? 2 : 1;
    int RT = (kCircThreads / ipr) * rpi;
    if (RT < rpi) RT = rpi;
    if (RT > 16) RT = 16;
    // three CTAs per SM (~75 KB each): as many stages as fit (bytes in flight hide HBM latency)
    const size_t budget = 75 * 1024;
    while (RT > rpi && circ_smem2(N, cls, nu, RT, 3) > budget) RT -= rpi;
    int S = 2;
    while (S < kMaxStages && circ_smem2(N, cls, nu, RT, S + 1) <= budget) ++S;
    return CircPlan{RT, S, circ_smem2(N, cls, nu, RT, S)};
}

template <int MODE, int CLS, bool UNIF, bool UBIAS, int NUCT>
static cudaError_t launch_circ_t(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st) {
    // paired rows where the register budget allows it without spills (nu == 1: the window streams)
    constexpr bool PAIR = MODE == MODE_PLAIN && UNIF && CLS == CLS_NU1;
    const CircPlan p = circ_plan(a.N, a.nu, PAIR);
    auto kern = layer_circ_kernel<MODE, CLS, UNIF, UBIAS, NUCT, PAIR>;
    int per_sm = 1;
    cudaError_t e = blocks_per_sm((const void*)kern, kCircThreads + 32, p.smem, &per_sm);
    if (e != cudaSuccess) return e;
    const int tiles = (max_rows + p.RT - 1) / p.RT;
    int grid = num_sms * per_sm;
    if (grid > tiles) grid = tiles;
    if (grid < 1) grid = 1;
    kern<<<grid, kCircThreads + 32, p.smem, st>>>(a, p.RT, p.S);
    return cudaGetLastError();
}

template <int MODE, int CLS, int NUCT>
static cudaError_t launch_circ_wb(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st) {
    const bool unif = a.wtab == nullptr;
    const bool ub = a.uniform_bias != 0;
    if (unif && ub) return launch_circ_t<MODE, CLS, true, true, NUCT>(a, max_rows, num_sms, st);
    if (unif) return launch_circ_t<MODE, CLS, true, false, NUCT>(a, max_rows, num_sms, st);
    if (ub) return launch_circ_t<MODE, CLS, false, true, NUCT>(a, max_rows, num_sms, st);
    return launch_circ_t<MODE, CLS, false, false, NUCT>(a, max_rows, num_sms, st);
}

template <int MODE>
static cudaError_t launch_circ_m(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st) {
    switch (circ_class(a.N, a.nu)) {
        case CLS_NU1: return launch_circ_wb<MODE, CLS_NU1, 0>(a, max_rows, num_sms, st);
        case CLS_Q32:  // compile-time nu for the SDGC strides: immediate shared-memory offsets
            if (a.nu == 32) return launch_circ_wb<MODE, CLS_Q32, 32>(a, max_rows, num_sms, st);
            if (a.nu == 128) return launch_circ_wb<MODE, CLS_Q32, 128>(a, max_rows, num_sms, st);
            if (a.nu == 512) return launch_circ_wb<MODE, CLS_Q32, 512>(a, max_rows, num_sms, st);
            return launch_circ_wb<MODE, CLS_Q32, 0>(a, max_rows, num_sms, st);
        default:
            if (a.nu == 32) return launch_circ_wb<MODE, CLS_GEN, 32>(a, max_rows, num_sms, st);
            return launch_circ_wb<MODE, CLS_GEN, 0>(a, max_rows, num_sms, st);
    }
}

cudaError_t launch_layer_circ(const LayerArgs& a, int mode, int max_rows, int num_sms, cudaStream_t st) {
    if (max_rows <= 0) return cudaSuccess;
    switch (mode) {
        case MODE_PLAIN: return launch_circ_m<MODE_PLAIN>(a, max_rows, num_sms, st);
        case MODE_CENTROID: return launch_circ_m<MODE_CENTROID>(a, max_rows, num_sms, st);
        default: return launch_circ_m<MODE_RESIDUAL>(a, max_rows, num_sms, st);
    }
}

}  // namespace snicit
