// kernels_circ_col.cu -- column-streaming circulant layer kernel for strided layers (nu >= 32), sm_100a.
//
// Same layer and arithmetic as kernels_circ.cu (Eq. 1; stored-order fma chain, reading
// R12), another data path.  With j = a*nu + c (Q = N/nu) a row is a Q x nu row-major matrix and a
// circulant layer of stride nu is a circular 1-D convolution of length K = 32 along a, independent for
// every column c:  y'[a][c] = sigma( sum_n w_n * y[(a + n) mod Q][c] + b ).  Column c is contiguous
// across c, so a warp owning 32 consecutive columns reads and writes whole 128-byte lines straight from
// and to global memory, and each thread slides its column's window through registers:
//   Q == 32  the window is the whole column: 32 loads, 32 outputs (rotations at compile time); the
//            next unit's 32 loads are issued before the current unit is computed (two register sets).
//   Q >= 64  a 64-register ring: input a lives in slot a & 63; after output a is produced, input a is
//            dead and the load of input a + 64 (mod Q) is issued into its slot, 64 outputs (2048 FMAs
//            of this warp) before it is used.  Only the 31 wrap-around inputs are read twice (L2).
// Every input element is read once from HBM and every output written once: 8 B per row-element, no
// shared memory, no staging copies.  Used for PLAIN-mode layers (pre-convergence, uncompressed path);
// a row's any-non-zero flag is OR-ed into flag_pos / flag_row (plain stores of 1, as the segmented
// kernel), and the caller's ordered compaction builds the next active list.
#include <cuda_runtime.h>

#include <type_traits>

#include "snicit_internal.cuh"

namespace snicit {

constexpr int kColThreads = 256;
constexpr int kColK = 32;

bool circ_col_supported(int N, int K, int nu) {
    if (K != kColK || nu < 32 || nu % 32 != 0 || N % nu != 0) return false;
    const int Q = N / nu;
    return Q >= 32 && Q % 32 == 0;
}

// per-n weights as a kernel parameter: the FMAs read them from the constant bank (no registers)
struct ColW {
    float w[kColK];
};

// NUCT: compile-time stride (0 = runtime a.nu) -- every load/store/bias offset of a chunk is then an
// immediate relative to one base pointer.  Q32: Q == 32 (whole-column units); else the 64-slot ring.
template <bool UNIF, bool UBIAS, bool Q32, int NUCT>
__global__ void __launch_bounds__(kColThreads, 2) layer_circ_col_kernel(LayerArgs a, const ColW cw) {
    const int N = a.N;
    const int nu = NUCT ? NUCT : a.nu;
    const int Q = N / nu;
    const unsigned G = (unsigned)nu >> 5;  // 32-column groups per row (compile-time with NUCT)
    // 32-bit unit indices (the launcher checks rows * G < 2^31): u / G is a shift for the SDGC strides
    const unsigned units = (unsigned)(*a.count) * G;
    const int lane = threadIdx.x & 31;
    const unsigned warp0 = (blockIdx.x * kColThreads + threadIdx.x) >> 5;
    const unsigned nwarps = (gridDim.x * kColThreads) >> 5;
    const float w0 = a.w0;
    const float b0 = UBIAS ? __ldg(a.bias) : 0.0f;
    const float ymax = a.ymax;

    if (blockIdx.x == 0 && threadIdx.x == 0 && a.zero_count) *a.zero_count = 0;  // next append counter

    // unit u = (list position, column group): offset of column c of the row
    auto unit_base = [&](unsigned u, int& pos, int& c) -> size_t {
        pos = (int)(u / G);
        c = (int)(u - (unsigned)pos * G) * 32 + lane;
        return (size_t)__ldg(a.rows + pos) * (size_t)N + (size_t)c;
    };
    // fused dead-row compaction (R23): rows with a non-zero output go to app_list (unordered, R24).
    // A row spans G warps: each counts in at row_ctr[pos] (+1, +65536 if it saw a non-zero) and the
    // last one decides, appends and clears the counter.  Appends are buffered one row per lane and
    // flushed with one atomic per 32 rows.
    int abuf = 0, nbuf = 0;
    auto flush = [&]() {
        int p0 = 0;
        if (lane == 0 && nbuf) p0 = atomicAdd(a.app_count, nbuf);
        p0 = __shfl_sync(0xffffffffu, p0, 0);
        if (lane < nbuf) a.app_list[p0 + lane] = abuf;
        nbuf = 0;
    };
    // constant-row mode (a.cmin, R26): rows whose outputs are all equal leave the list for the
    // constant list (row, value, layer); the warps of a row combine (min, max) at cmin/cmax[pos]
    auto push_const = [&](int row, float v, int layer) {
        const int p = atomicAdd(a.ccount, 1);
        a.clist[p] = row;
        a.cval[p] = v;
        a.clayer[p] = layer;
    };
    // Constant-row mode walks the units row-major per warp (all G column groups of a row in one warp,
    // see nextu), so a row's output range is combined in registers and decided by that warp alone.
    const bool rowmajor = a.cmin != nullptr;
    float rmx = 0.0f, rmn = ymax;  // running range of the current row (constant-row mode)
    auto flag = [&](int pos, size_t base, float mx, float mn, bool last) {
        if (rowmajor) {
            rmx = fmaxf(rmx, mx);
            rmn = fminf(rmn, mn);
            if (!last) return;
#pragma unroll
            for (int d = 16; d; d >>= 1) {
                rmx = fmaxf(rmx, __shfl_xor_sync(0xffffffffu, rmx, d));
                rmn = fminf(rmn, __shfl_xor_sync(0xffffffffu, rmn, d));
            }
            const unsigned umn = __float_as_uint(rmn + 0.0f), umx = __float_as_uint(rmx + 0.0f);  // -0 -> +0
            rmx = 0.0f;
            rmn = ymax;
            const int row = (int)(base / (size_t)N);
            if (umn == umx) {
                const float v = __uint_as_float(umn);
                if (lane == 0 && !(v == 0.0f && a.dead_drop)) push_const(row, v, a.layer);
            } else if (__uint_as_float(umn) >= a.thr_hi) {  // range prediction (R30): YMAX at t
                if (lane == 0) push_const(row, ymax, a.thr_layer);
            } else if (__uint_as_float(umx) <= a.thr_lo) {  // R30: zero at t (dead, or a constant zero row)
                if (lane == 0 && !a.thr_dead) push_const(row, 0.0f, a.thr_layer);
            } else {
                if (lane == nbuf) abuf = row;
                if (++nbuf == 32) flush();
            }
            return;
        }
        const bool nz = __any_sync(0xffffffffu, mx != 0.0f);
        if (a.app_list) {
            int app = 0;
            if (lane == 0) {
                if (G == 1) {
                    app = nz;
                } else {
                    const int old = atomicAdd(a.row_ctr + pos, 1 + (nz ? 65536 : 0));
                    if ((old & 0xffff) == G - 1) {
                        app = nz || (old >> 16) != 0;
                        a.row_ctr[pos] = 0;
                    }
                }
            }
            if (__shfl_sync(0xffffffffu, app, 0)) {
                if (lane == nbuf) abuf = (int)(base / (size_t)N);
                if (++nbuf == 32) flush();
            }
        } else if (nz && lane == 0) {
            if (a.flag_pos) a.flag_pos[pos] = 1;
            if (a.flag_row) a.flag_row[base / (size_t)N] = 1;
        }
    };
    // output epilogue: Eq. 1 bias + sigma (Table 2), store, running max / min for the row flags
    auto emit = [&](float acc, float* dst, const float* bsrc, float& mx, float& mn) {
        const float bq = UBIAS ? b0 : __ldg(bsrc);
        const float v = sigma(acc + bq, ymax);
        *dst = v;
        mx = fmaxf(mx, v);
        mn = fminf(mn, v);
    };

    // unit order: round-robin over warps, or (constant-row mode) row-major: warp w takes rows w,
    // w + nwarps, ... and within a row its G column groups in order
    const unsigned u_first = rowmajor ? warp0 * G : warp0;
    auto nextu = [&](unsigned u) -> unsigned {
        if (!rowmajor) return u + nwarps;
        return (u % G == G - 1) ? (u / G + nwarps) * G : u + 1;
    };
    auto is_last = [&](unsigned u) -> bool { return u % G == G - 1; };

    if constexpr (Q32) {
        // ---------------------------------------------------------------- Q == 32: whole column
        auto load = [&](float (&R)[32], size_t base) {
            const float* src = a.yin + base;
#pragma unroll
            for (int i = 0; i < 32; ++i) R[i] = src[i * nu];
        };
        auto compute = [&](const float (&R)[32], size_t base, int c, int pos, bool last) {
            float* dst = a.yout + base;
            const float* bsrc = a.bias + c;
            float mx = 0.0f, mn = ymax;
#pragma unroll
            for (int m = 0; m < 32; ++m) {
                float acc = 0.0f;
#pragma unroll
                for (int n = 0; n < kColK; ++n) acc = fmaf(R[(m + n) & 31], UNIF ? w0 : cw.w[n], acc);
                emit(acc, dst + m * nu, bsrc + m * nu, mx, mn);
            }
            flag(pos, base, mx, mn, last);
        };
        float RA[32], RB[32];
        unsigned u = u_first;
        int posA = 0, cA = 0, posB = 0, cB = 0;
        size_t bA = 0, bB = 0;
        if (u < units) {
            bA = unit_base(u, posA, cA);
            load(RA, bA);
        }
        while (u < units) {
            const unsigned u2 = nextu(u);
            if (u2 < units) {
                bB = unit_base(u2, posB, cB);
                load(RB, bB);
            }
            compute(RA, bA, cA, posA, is_last(u));
            if (u2 >= units) break;
            const unsigned u3 = nextu(u2);
            if (u3 < units) {
                bA = unit_base(u3, posA, cA);
                load(RA, bA);
            }
            compute(RB, bB, cB, posB, is_last(u2));
            u = u3;
        }
    } else {
        // ---------------------------------------------------------------- Q >= 64: 64-slot ring
        // Input a lives in slot a & 63 (a = 0 .. Q + 30, inputs a >= Q being a - Q again).  A chunk is
        // 32 outputs a0 + m from slots (SB + m + n) & 63 (SB = a0 & 63: a compile-time 0 or 32); after
        // output a0 + m its slot SB + m is dead and, for m < nload, is refilled from ld[m * nu] with
        // input a0 + 64 + m.  One loop body (two chunks) serves every step, tail included: the code
        // stays small enough for the instruction cache (fully unrolled tails thrashed it).
        float R[64];
        auto chunk = [&](auto sb_tag, const float* ld, int nload, float* st, const float* bs, float& mx, float& mn) {
            constexpr int SB = decltype(sb_tag)::value;
#pragma unroll
            for (int m = 0; m < 32; ++m) {
                float acc = 0.0f;
#pragma unroll
                for (int n = 0; n < kColK; ++n) acc = fmaf(R[(SB + m + n) & 63], UNIF ? w0 : cw.w[n], acc);
                emit(acc, st + m * nu, bs + m * nu, mx, mn);
                if (m < nload) R[SB + m] = ld[m * nu];
            }
        };
        // offset of the 32-block of inputs starting at a (a multiple of 32, a < 2Q): never straddles Q
        auto blk = [&](int x) -> size_t { return (size_t)(x < Q ? x : x - Q) * nu; };
        // refills of the block starting at input x: inputs up to Q + 30 are needed
        auto nld = [&](int x) -> int { return min(32, max(0, Q + 31 - x)); };
        using I0 = std::integral_constant<int, 0>;
        using I32 = std::integral_constant<int, 32>;
        for (unsigned u = u_first; u < units; u = nextu(u)) {
            int pos, c;
            const size_t base = unit_base(u, pos, c);
            const float* src = a.yin + base;
            float* dst = a.yout + base;
            const float* bsrc = a.bias + c;
#pragma unroll
            for (int i = 0; i < 64; ++i) R[i] = src[i * nu];  // inputs 0..63 (Q >= 64)
            float mx = 0.0f, mn = ymax;
            for (int a0 = 0; a0 < Q; a0 += 64) {
                const size_t o0 = (size_t)a0 * nu;
                chunk(I0(), src + blk(a0 + 64), nld(a0 + 64), dst + o0, bsrc + o0, mx, mn);
                if (a0 + 32 < Q) {
                    const size_t o1 = o0 + 32 * (size_t)nu;
                    chunk(I32(), src + blk(a0 + 96), nld(a0 + 96), dst + o1, bsrc + o1, mx, mn);
                }
            }
            flag(pos, base, mx, mn, is_last(u));
        }
    }
    if (a.app_list) flush();
}

template <bool UNIF, bool UBIAS, bool Q32, int NUCT>
static cudaError_t launch_col_t(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st) {
    auto kern = layer_circ_col_kernel<UNIF, UBIAS, Q32, NUCT>;
    int per_sm = 1;
    cudaError_t e = blocks_per_sm((const void*)kern, kColThreads, 0, &per_sm);
    if (e != cudaSuccess) return e;
    const long long units = (long long)max_rows * (a.nu / 32);
    if (units + (long long)num_sms * 64 >= (1LL << 31)) return cudaErrorInvalidValue;  // 32-bit unit ids
    long long grid = (long long)num_sms * per_sm;
    const long long need = (units + kColThreads / 32 - 1) / (kColThreads / 32);
    if (grid > need) grid = need;
    if (grid < 1) grid = 1;
    // row-major unit walk (constant-row mode) steps past the last unit by up to nwarps * G
    if (units + grid * (kColThreads / 32) * (long long)(a.nu / 32) >= (1LL << 31)) return cudaErrorInvalidValue;
    ColW cw{};
    if (!UNIF)
        for (int n = 0; n < kColK; ++n) cw.w[n] = a.wtab_host[n];
    kern<<<(int)grid, kColThreads, 0, st>>>(a, cw);
    return cudaGetLastError();
}

template <bool Q32, int NUCT>
static cudaError_t launch_col_q(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st) {
    const bool unif = a.wtab == nullptr, ub = a.uniform_bias != 0;
    if (unif && ub) return launch_col_t<true, true, Q32, NUCT>(a, max_rows, num_sms, st);
    if (unif) return launch_col_t<true, false, Q32, NUCT>(a, max_rows, num_sms, st);
    if (ub) return launch_col_t<false, true, Q32, NUCT>(a, max_rows, num_sms, st);
    return launch_col_t<false, false, Q32, NUCT>(a, max_rows, num_sms, st);
}

cudaError_t launch_layer_circ_col(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st) {
    if (max_rows <= 0) return cudaSuccess;
    if (a.N / a.nu == 32) {  // SDGC: N = 4096 / 16384 / 65536 -> nu = 128 / 512 / 2048
        if (a.nu == 128) return launch_col_q<true, 128>(a, max_rows, num_sms, st);
        if (a.nu == 512) return launch_col_q<true, 512>(a, max_rows, num_sms, st);
        if (a.nu == 2048) return launch_col_q<true, 2048>(a, max_rows, num_sms, st);
        return launch_col_q<true, 0>(a, max_rows, num_sms, st);
    }
    if (a.nu == 32) return launch_col_q<false, 32>(a, max_rows, num_sms, st);  // every SDGC size
    if (a.nu == 1024) return launch_col_q<false, 1024>(a, max_rows, num_sms, st);  // N = 65536
    return launch_col_q<false, 0>(a, max_rows, num_sms, st);
}

}  // namespace snicit
