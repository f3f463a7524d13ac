// kernels_pre_fused.cu -- row-resident pre-convergence phase (a1), sm_100a.
//
// Eq. 1 is applied to every batch row independently, layer after layer, so a row can stay
// in shared memory for all t pre-convergence layers: one CTA loads a row from HBM once (TMA bulk
// copy), evaluates layers 0..t-1 ping-ponging between two shared-memory buffers, and writes Y(t) once.
// HBM traffic drops from 8 B per row-element per layer to 8 B per row-element per t layers; the kernel
// is bound by the FP32 FMA pipe (32 fma per output, exact stored-order chains, R12) instead of HBM.
//
// Per layer (all layers circulant, K = 32 taps, uniform weight w0, uniform bias b0 -- the SDGC
// RadiX layers): T = N/32 threads, each evaluating two work items at once with packed
// fma.rn.f32x2 (FFMA2: per-lane RN fmas, bit-identical to fmaf, R17) -- two items of the SAME row and
// layer, so the pair never diverges.  Stride classes:
//   NU1  nu == 1: N = 17T + 15T: thread i owns outputs [17i, 17i + 17) and [17T + 15i, 17T + 15i + 15)
//        (odd lane strides: conflict-free LDS; exact tiling), paired for 15 outputs.
//   STR  nu >= 32 with Q = N/nu >= 64: item (c, a0) = outputs (a0 + m)*nu + c, m < 16, window of 47
//        inputs of residue class c; lanes on consecutive c (conflict-free); the pair is (c, a0) and
//        (c, a0 + Q/2), i.e. base offsets b and b + N/2.
//   Q32  nu == N/32: a thread owns residue class c (T == nu) -- 32 inputs, the two items are
//        a0 = 0 and a0 = 16 and every rotation is compile-time.
// Windows never wrap: every buffer carries a circular halo (a copy of the row head, H floats: 64 for
// NU1, and 31*nu of STR layers); each layer writes outputs q < H twice.
//
// Constant rows (R26, exact): a circulant layer with uniform weight and bias maps a row whose elements
// are all equal to v to the constant row sigma(chain(v) + b0) -- every output evaluates the same
// stored-order chain on the same values (the R25 argument of the post phase).  After each layer the
// CTA tests "all outputs equal"; a constant row is then carried by one scalar
// chain per remaining layer and written with plain vector stores.  The test costs no extra barrier:
// warps vote on their outputs and publish (vote, value) before the layer's barrier.  An all-zero row is dead (R23) when
// every later bias is <= 0: it leaves without a write.  Survivors are appended (unordered, R24) to the
// active list at t.  Rows are scheduled dynamically (one atomic per row).
#include <cuda_runtime.h>

#include <cmath>
#include <cstring>

#include "snicit_internal.cuh"

namespace snicit {

constexpr int kPfM1 = 17;  // NU1 outputs per item
constexpr int kPfM = 16;   // STR / Q32 outputs per item
constexpr int kPfSurv = 32;  // survivor batch per CTA
constexpr int kPfW = kPfM + 31;
constexpr int kPfConstChunk = 1024;  // floats per constant-row TMA store (NB == 3)

typedef unsigned long long u64;

// ---------------------------------------------------------------------------- layer bodies
// nu == 1: N = 32T = 17T + 15T, so thread i owns item 1 = outputs [17i, 17i + 17) and item 2 =
// [17T + 15i, 17T + 15i + 15): both lane strides odd (conflict-free LDS), the row tiled exactly (no
// idle lanes, no outputs past N).  Outputs 0..14 of both items are FFMA2 pairs; item 1's outputs 15,
// 16 are scalar chains on the low halves (half the FMA-pipe cycles of a half-used pair).  Windows read
// up to N + 30 (halo); the head outputs q < H are also written to the halo.
template <int T>
__device__ __forceinline__ void pf_body_nu1(const float* __restrict__ in, float* __restrict__ out, float w0, float b0,
                                            float ymax, int H, float& mn, float& mx) {
    constexpr int N = 32 * T;
    constexpr int M2 = 15;           // item 2 outputs
    constexpr int W2N = M2 + 31;     // paired window (46)
    const int i1 = threadIdx.x;
    const float* s1 = in + kPfM1 * i1;
    const float* s2 = in + kPfM1 * T + M2 * i1;
    u64 R[W2N];
#pragma unroll
    for (int i = 0; i < W2N; ++i) R[i] = f2_pack(s1[i], s2[i]);
    const float e46 = s1[W2N], e47 = s1[W2N + 1];  // item 1's window tail
    const u64 W2 = f2_pack(w0, w0), B2 = f2_pack(b0, b0);
    float o1s[kPfM1];
    float* d1 = out + kPfM1 * i1;
    float* d2 = out + kPfM1 * T + M2 * i1;
#pragma unroll
    for (int m = 0; m < M2; ++m) {
        u64 acc = 0ull;
#pragma unroll
        for (int n = 0; n < 32; ++n) acc = f2_fma(R[m + n], W2, acc);
        float z1, z2;
        f2_unpack(f2_add(acc, B2), z1, z2);
        const float o1 = sigma(z1, ymax), o2 = sigma(z2, ymax);
        d1[m] = o1;
        d2[m] = o2;
        o1s[m] = o1;
        mn = fminf(mn, fminf(o1, o2));
        mx = fmaxf(mx, fmaxf(o1, o2));
    }
#pragma unroll
    for (int m = M2; m < kPfM1; ++m) {  // item 1 only: scalar chains on the low halves
        float acc = 0.0f;
#pragma unroll
        for (int n = 0; n < 32; ++n) {
            float x;
            if (m + n < W2N) {
                float hi;
                f2_unpack(R[m + n], x, hi);
            } else {
                x = (m + n == W2N) ? e46 : e47;
            }
            acc = fmaf(x, w0, acc);
        }
        const float o1 = sigma(acc + b0, ymax);
        d1[m] = o1;
        o1s[m] = o1;
        mn = fminf(mn, o1);
        mx = fmaxf(mx, o1);
    }
    if (kPfM1 * i1 < H) {  // head outputs -> halo (item 2 starts at 17T > H)
#pragma unroll
        for (int m = 0; m < kPfM1; ++m)
            if (kPfM1 * i1 + m < H) out[N + kPfM1 * i1 + m] = o1s[m];
    }
}

// NU > 0: compile-time stride; NU == 0: runtime nu.  Item 1 (a0 <= Q/2 - 16) never wraps for Q >= 64;
// item 2 (a-rows a0 + Q/2 + i) wraps: HALO -> the buffers carry H >= 31*nu floats of circular halo;
// otherwise its a-row index is taken mod Q (Q a power of two: a mask), which keeps the smem small.
template <int T, int NU, bool HALO>
__device__ __forceinline__ void pf_body_str(const float* __restrict__ in, float* __restrict__ out, int nu_rt, float w0,
                                            float b0, float ymax, int H, float& mn, float& mx) {
    constexpr int N = 32 * T;
    const int nu = NU ? NU : nu_rt;
    const int Q = N / nu;
    const int c = (int)threadIdx.x % nu;
    const int a0 = ((int)threadIdx.x / nu) * kPfM;
    const int base = a0 * nu + c;
    const float* s = in + base;
    u64 R[kPfW];
    if constexpr (HALO) {
#pragma unroll
        for (int i = 0; i < kPfW; ++i) R[i] = f2_pack(s[i * nu], s[i * nu + N / 2]);
    } else {
        const float* sc = in + c;
        const int k2 = a0 + Q / 2;
#pragma unroll
        for (int i = 0; i < kPfW; ++i) R[i] = f2_pack(s[i * nu], sc[((k2 + i) & (Q - 1)) * nu]);
    }
    const u64 W2 = f2_pack(w0, w0), B2 = f2_pack(b0, b0);
#pragma unroll
    for (int m = 0; m < kPfM; ++m) {
        u64 acc = 0ull;
#pragma unroll
        for (int n = 0; n < 32; ++n) acc = f2_fma(R[m + n], W2, acc);
        float z1, z2;
        f2_unpack(f2_add(acc, B2), z1, z2);
        const float o1 = sigma(z1, ymax), o2 = sigma(z2, ymax);
        const int q1 = base + m * nu, q2 = q1 + N / 2;
        out[q1] = o1;
        out[q2] = o2;
        if (q1 < H) out[N + q1] = o1;
        if (HALO && q2 < H) out[N + q2] = o2;
        mn = fminf(mn, fminf(o1, o2));
        mx = fmaxf(mx, fmaxf(o1, o2));
    }
}

template <int T>
__device__ __forceinline__ void pf_body_q32(const float* __restrict__ in, float* __restrict__ out, float w0, float b0,
                                            float ymax, int H, float& mn, float& mx) {
    constexpr int N = 32 * T;
    constexpr int nu = T;  // Q == 32
    const int c = threadIdx.x;
    float x[32];
#pragma unroll
    for (int k = 0; k < 32; ++k) x[k] = in[k * nu + c];
    u64 P[32];  // P[k] = (x[k], x[k + 16 mod 32]): item a0 = 0 in the low lane, a0 = 16 in the high lane
#pragma unroll
    for (int k = 0; k < 32; ++k) P[k] = f2_pack(x[k], x[(k + 16) & 31]);
    const u64 W2 = f2_pack(w0, w0), B2 = f2_pack(b0, b0);
#pragma unroll
    for (int m = 0; m < kPfM; ++m) {
        u64 acc = 0ull;
#pragma unroll
        for (int n = 0; n < 32; ++n) acc = f2_fma(P[(m + n) & 31], W2, acc);
        float z1, z2;
        f2_unpack(f2_add(acc, B2), z1, z2);
        const float o1 = sigma(z1, ymax), o2 = sigma(z2, ymax);
        const int q1 = m * nu + c, q2 = q1 + 16 * nu;
        out[q1] = o1;
        out[q2] = o2;
        if (q1 < H) out[N + q1] = o1;
        if (q2 < H) out[N + q2] = o2;
        mn = fminf(mn, fminf(o1, o2));
        mx = fmaxf(mx, fmaxf(o1, o2));
    }
}

// Class-sum bounds of a Q32 layer (R31): thread c owns residue class c, and every output of the class is a
// chain over the same 32 elements (a rotation of them), so one pass of directed-rounding sums bounds all
// 32 outputs of the class before any of them is evaluated.  Inputs are >= 0 (outputs of sigma), w0 >= 0:
// each RN step of a chain satisfies y (1 - u) - 2^-150 <= RN(y) <= y (1 + u) + 2^-150 (u = 2^-24), so a
// chain in any order lies in [(1 - u)^32 S - 32 2^-150, (1 + u)^32 S + 32 2^-150], S = sum x w0 exactly,
// bracketed by the round-down / round-up chains; (1 - u)^32 >= 1 - 2^-19, (1 + u)^32 <= 1 + 2^-18.  The
// bias add and sigma are monotone, so sigma(RD(lo + b0)) <= y <= sigma(RU(hi + b0)) for every output y.
template <int T>
__device__ __forceinline__ void pf_q32_bounds(const float* __restrict__ in, float w0, float b0, float ymax,
                                              float& ylo, float& yhi) {
    constexpr int nu = T;
    const int c = threadIdx.x;
    float slo = 0.0f, shi = 0.0f;
#pragma unroll
    for (int k = 0; k < 32; ++k) {
        const float x = in[k * nu + c];
        slo = __fmaf_rd(x, w0, slo);
        shi = __fmaf_ru(x, w0, shi);
    }
    const float lo = __fsub_rd(__fmul_rd(slo, 1.0f - 0x1p-19f), 0x1p-140f);
    const float hi = __fadd_ru(__fmul_ru(shi, 1.0f + 0x1p-18f), 0x1p-140f);
    ylo = sigma(__fadd_rd(lo, b0), ymax);
    yhi = sigma(__fadd_ru(hi, b0), ymax);
}

// R34 (exact): bounds of a stride-1 layer's outputs before it is evaluated.  Output q = sigma(chain over
// x[q..q+31] + b0); with inputs >= 0 and w0 >= 0 the chain in any order lies in [(1 - 2^-19) S w0 -
// 2^-140, (1 + 2^-18) S w0 + 2^-140] (R31), S = the exact window sum.  A thread bounds S for its item-1
// and item-2 windows (pf_body_nu1's mapping: conflict-free loads) by sliding directed sums -- lo' =
// RD(RD(lo + x_new) - x_old) <= S' whenever lo <= S (and the RU mirror) -- and returns the min / max
// output bounds over its windows.
template <int T>
__device__ __forceinline__ void pf_nu1_bounds(const float* __restrict__ in, float w0, float b0, float ymax,
                                              float& ylo, float& yhi) {
    constexpr int M2 = 15;
    const int i1 = threadIdx.x;
    float smin = __int_as_float(0x7f800000), smax = 0.0f;
#pragma unroll
    for (int it = 0; it < 2; ++it) {
        const float* src = it == 0 ? in + kPfM1 * i1 : in + kPfM1 * T + M2 * i1;
        const int M = it == 0 ? kPfM1 : M2;
        float lo = 0.0f, hi = 0.0f;
#pragma unroll
        for (int n = 0; n < 32; ++n) {
            const float x = src[n];
            lo = __fadd_rd(lo, x);
            hi = __fadd_ru(hi, x);
        }
        smin = fminf(smin, lo);
        smax = fmaxf(smax, hi);
#pragma unroll
        for (int m = 1; m < kPfM1; ++m) {
            if (m < M) {
                const float xn = src[m + 31], xo = src[m - 1];
                lo = __fsub_rd(__fadd_rd(lo, xn), xo);
                hi = __fsub_ru(__fadd_ru(hi, xn), xo);
                smin = fminf(smin, lo);
                smax = fmaxf(smax, hi);
            }
        }
    }
    smin = fmaxf(smin, 0.0f);  // S >= 0
    const float clo = __fsub_rd(__fmul_rd(__fmul_rd(smin, w0), 1.0f - 0x1p-19f), 0x1p-140f);
    const float chi = __fadd_ru(__fmul_ru(__fmul_ru(smax, w0), 1.0f + 0x1p-18f), 0x1p-140f);
    ylo = sigma(__fadd_rd(clo, b0), ymax);
    yhi = sigma(__fadd_ru(chi, b0), ymax);
}

// R32: layer 0 of stride 1 as a table lookup when the row holds zeros and one value c (checked here for
// fp32 rows; packed rows are binary with c = one).  Warp w owns the words j = 32 w .. 32 w + 31 of the
// row's bitmap (bit b of word j = element 32 j + b != 0; lane i holds word 32 w + i, built by one ballot
// per word for fp32 rows or read from the packed row) and lane i the outputs q = 32 j + e of its word j:
// window q .. q + 31 = bits e .. e + 31 of (word j + 1 : word j), k = popc of it, output tab[k] (the
// warp's copy of tab[k] = sigma(chain of k fmas of c from +0, + b0), k = 0..32, in shared memory).  The
// lanes walk e = (b + lane) mod 32 so the stores of one step hit 32 different banks.  Returns false
// (nothing written) for a row with two different non-zero values, a NaN or c < 0.
__device__ __forceinline__ float max_nan(float a, float b) {
    float r;
    asm("max.NaN.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b));
    return r;
}
constexpr int kPfTabStride = 40;  // floats per warp table (33 used)
template <int T>
__device__ __forceinline__ bool pf_popc_layer0(const float* __restrict__ in, float* __restrict__ out,
                                               const uint32_t* pwords, float one, float w0, float b0, float ymax,
                                               int H, unsigned* s_red, float* s_tabw, float& mn, float& mx) {
    constexpr int N = 32 * T, W = N / 32, kWarps = T / 32;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int j0 = warp * 32;  // W / kWarps == 32 words per warp
    uint32_t wl, wnext;
    float c = one;
    if (pwords) {
        wl = pwords[j0 + lane];
        wnext = pwords[(j0 + 32) & (W - 1)];
    } else {
        float nzmin = __int_as_float(0x7f800000), nzmax = -__int_as_float(0x7f800000);
        wl = 0u;
        const float* src = in + j0 * 32 + lane;
#pragma unroll 8
        for (int i = 0; i < 32; ++i) {
            const float x = src[i * 32];
            const bool nz = x != 0.0f;
            const uint32_t bw = __ballot_sync(0xffffffffu, nz);
            wl = lane == i ? bw : wl;
            nzmin = fminf(nzmin, nz ? x : __int_as_float(0x7f800000));
            nzmax = max_nan(nzmax, x);
        }
        wnext = __ballot_sync(0xffffffffu, in[((j0 + 32) & (W - 1)) * 32 + lane] != 0.0f);
#pragma unroll
        for (int d = 16; d; d >>= 1) {
            nzmin = fminf(nzmin, __shfl_xor_sync(0xffffffffu, nzmin, d));
            nzmax = max_nan(nzmax, __shfl_xor_sync(0xffffffffu, nzmax, d));
        }
        if (lane == 0) {
            s_red[warp] = __float_as_uint(nzmin);
            s_red[kWarps + warp] = __float_as_uint(nzmax);
        }
        __syncthreads();
        float gmin = __int_as_float(0x7f800000), gmax = -__int_as_float(0x7f800000);
#pragma unroll
        for (int w = 0; w < kWarps; ++w) {
            gmin = fminf(gmin, __uint_as_float(s_red[w]));
            gmax = max_nan(gmax, __uint_as_float(s_red[kWarps + w]));
        }
        __syncthreads();  // s_red read by every thread before it is reused
        // two-valued: every non-zero equals gmax (> 0); all zero: gmax = 0, every count 0
        if (gmax == 0.0f) c = 0.0f;
        else if (gmin == gmax && gmax > 0.0f) c = gmax;
        else return false;
    }
    float* tw = s_tabw + warp * kPfTabStride;
    {
        float acc = 0.0f;
        for (int n = 0; n < lane; ++n) acc = fmaf(c, w0, acc);
        tw[lane] = sigma(acc + b0, ymax);
        const float acc31 = __shfl_sync(0xffffffffu, acc, 31);
        if (lane == 0) tw[32] = sigma(fmaf(c, w0, acc31) + b0, ymax);
    }
    __syncwarp();
    const uint32_t wn = __shfl_down_sync(0xffffffffu, wl, 1);
    const uint32_t wj1 = lane < 31 ? wn : wnext;
    float* dst = out + (j0 + lane) * 32;
    const int qb = (j0 + lane) * 32;
    const bool halo = j0 * 32 < H;  // warp-uniform
    int kmin = 32, kmax = 0;
#pragma unroll 8
    for (int b = 0; b < 32; ++b) {
        const int e = (b + lane) & 31;
        const int k = __popc(__funnelshift_r(wl, wj1, e));
        const float o = tw[k];
        dst[e] = o;
        if (halo && qb + e < H) dst[N + e] = o;
        kmin = min(kmin, k);
        kmax = max(kmax, k);
    }
    // tab is monotone in k (chains of one value c >= 0, sigma monotone): the range is tab[kmin], tab[kmax]
    kmin = __reduce_min_sync(0xffffffffu, kmin);
    kmax = __reduce_max_sync(0xffffffffu, kmax);
    mn = fminf(mn, tw[kmin]);
    mx = fmaxf(mx, tw[kmax]);
    return true;
}

// STR wrap handling: a 31*nu halo, or (kPfStrHalo = false) the a-row index mod Q
template <int T>
constexpr bool kPfStrHalo = true;  // measured: the masked form (H = 64, 6 CTAs/SM at N = 4096) is slower
bool pre_fused_str_halo(int N) { return kPfStrHalo<128> || N < 0; }

// row buffers: two (ping-pong) and, when one CTA fills the SM anyway (N = 16384), a third that receives
// the next row while this one computes (otherwise the next row is only prefetched into L2)
template <int T>
constexpr int kPfBufs = T >= 512 ? 3 : 2;

template <int T>
struct PfCfg {
    static constexpr int kMinBlocks = T <= 32 ? 16 : (T <= 64 ? 8 : (T <= 128 ? 4 : (T <= 256 ? 2 : 1)));
};

// ---------------------------------------------------------------------------- the kernel
// Layer descriptors travel in the kernel's parameter space (constant bank).  When every layer has the
// same weight it is read at a constant offset, so the FFMA2 weight operand is a uniform register
// (fewer register-file reads than a per-thread copy: measured +5% on the Q32 / STR bodies).
struct PfLayerParam {
    float w0, b0;
    int nu;
    int flags;  // cls | dead_next << 4 | ymax_fixed << 5 | ymax fixed for all later layers < t << 6
};
// range prediction (R30): thr_hi[k-1] = least m with out^k(m) == YMAX, thr_lo[k-1] = greatest m with
// out^k(m) == 0, out(m) = sigma(chain(m) + b0) the layers' map of a constant row (host-evaluated with the
// kernels' fma order); k > kPfThr uses entry kPfThr (thr_hi non-increasing and thr_lo non-decreasing in
// k, so the shorter horizon is the stricter test)
constexpr int kPfThr = kRangeK;
struct PreFusedParams {
    PreFusedArgs a;
    float thr_hi[kPfThr], thr_lo[kPfThr];
    PfLayerParam L[kPfMaxLayers];
};
static_assert(sizeof(PreFusedParams) <= 32764, "kernel parameter space");

// GENSTR: the network has STR layers with nu != 32 (runtime-stride body compiled in); WUNI: every
// layer < t has the same weight
template <int T, bool GENSTR, bool WUNI>
__global__ void __launch_bounds__(T, PfCfg<T>::kMinBlocks) pre_fused_kernel(const __grid_constant__ PreFusedParams p) {
    const PreFusedArgs& a = p.a;
    constexpr int N = 32 * T;
    extern __shared__ __align__(128) unsigned char smem[];
    const int H = a.H;
    const int S = N + H;  // buffer stride (floats): row + circular halo
    constexpr int NB = kPfBufs<T>;
    float* const buf = reinterpret_cast<float*>(smem);  // NB buffers of S floats
    uint64_t* bar = reinterpret_cast<uint64_t*>(buf + NB * S);  // [2] row loads, alternating per row
    int* s_pos = reinterpret_cast<int*>(bar + 2);               // [0] first row, [2 + (k & 1)] next row
    constexpr int kWarps = T / 32;
    unsigned* s_vmn = reinterpret_cast<unsigned*>(s_pos + 4);  // [2][kWarps] per-warp output minimum (bits)
    unsigned* s_vmx = s_vmn + 2 * kWarps;                      // [2][kWarps] per-warp output maximum
    unsigned* s_bmn = s_vmx + 2 * kWarps;                      // [kWarps] Q32 class-sum bounds (R31)
    unsigned* s_bmx = s_bmn + 2 * kWarps;                      //   (slots of 2 kWarps: s_bits stays 16-B aligned)
    const int tid = threadIdx.x;
    const int count = *a.count;
    if (tid == 0) {
        mbar_init(&bar[0], 1);
        mbar_init(&bar[1], 1);
        fence_proxy_async_smem();
        s_pos[0] = atomicAdd(a.work, 1);
    }
    __syncthreads();
    int pos = s_pos[0];
    // one row (and its circular halo: a second copy of the row head) -> buffer `dst`, completion on `b`
    unsigned* s_red = s_bmx + 2 * kWarps;  // [4 kWarps] R32's fp32-row reduction (its own: no row-end barrier)
    uint32_t* s_bits = reinterpret_cast<uint32_t*>(s_red + 4 * kWarps);  // [2][N/32] packed rows (a.ybits)
    int* s_surv = reinterpret_cast<int*>(s_bits + 2 * (N / 32));       // [kPfSurv] rows alive at t, batched
    // NB == 3 (one CTA per SM): 4 KB rows of zeros and of YMAX, the sources of the TMA bulk stores that
    // write dead rows and constant-YMAX rows (16 bulk copies issued by one thread instead of N/4 vector
    // stores from every warp); written once, never modified
    float* s_tabw = reinterpret_cast<float*>(s_surv + kPfSurv);  // [kWarps][kPfTabStride] R32 tables
    float* s_cz = s_tabw + kWarps * kPfTabStride;
    float* s_cy = s_cz + kPfConstChunk;
    bool prev_res = false;  // (tid 0, NB == 3) the previous row ended with a TMA store of a row buffer
    int nsurv = 0;                                                     // (tid 0) entries in s_surv
    // one atomic per kPfSurv survivors (an atomic whose result is waited on stalls the whole CTA at the
    // next barrier; per row that was ~1 us)
    auto flush_surv = [&](bool force) {
        if (tid == 0 && nsurv > 0 && (force || nsurv == kPfSurv)) {
            const int p0 = atomicAdd(a.app_count, nsurv);
            for (int i = 0; i < nsurv; ++i) a.app_list[p0 + i] = s_surv[i];
            nsurv = 0;
        }
    };
    auto issue_load = [&](int p_, float* dst, uint64_t* b, int slot) {
        const size_t r_ = (size_t)__ldg(a.rows + p_);
        if (a.ready) {  // streamed upload: wait until the copy engine has delivered this row's chunk
            // geometric chunks: chunk c holds rows [b (2^c - 1), b (2^(c+1) - 1)), b = ready_rows
            const int* f = a.ready + (31 - __clz((int)(r_ / a.ready_rows) + 1));
            while (ld_acquire_gpu(f) == 0) __nanosleep(256);
            fence_proxy_async_global();
        }
        if (a.ybits) {  // packed binary row: N/8 bytes
            mbar_arrive_expect_tx(b, (uint32_t)(N / 8));
            bulk_g2s(s_bits + slot * (N / 32), a.ybits + r_ * (N / 32), N / 8, b);
        } else {
            const float* g = a.yin + r_ * N;
            mbar_arrive_expect_tx(b, (uint32_t)(S * 4));
            bulk_g2s(dst, g, N * 4, b);
            bulk_g2s(dst + N, g, H * 4, b);
        }
    };
    if (NB == 3) {
        for (int i = tid; i < kPfConstChunk; i += T) {
            s_cz[i] = 0.0f;
            s_cy[i] = a.ymax;
        }
        fence_proxy_async_smem();
        __syncthreads();
    }
    int i_in = 0, i_out = 1, i_pf = 2;  // buffer roles (NB == 3: i_pf receives the next row)
    // No CTA barrier at the row end.  The next row's first layer writes only the buffer its predecessor's
    // last layer READ (finished before that layer's barrier), its position slot (claimed a row ahead,
    // published at the row start) differs from the one being read, the range slots use a running
    // layer-instance parity (gl), R32 reduces through its own scratch, and a row buffer is reloaded only
    // after its TMA store was read -- so warps may start the next row while warp 0 finishes the bookkeeping
    // (round 2 (r02c))
    int gl = 0;  // evaluated layer instances (range slot parity)
    uint32_t ph = 0;                    // phase bit of bar[0], bar[1]
    if (NB == 3 && tid == 0 && pos < count) issue_load(pos, buf, &bar[0], 0);
    int np = 0;  // tid 0: the next row's list position
    // the position after that, claimed one row ahead so the atomic's latency is never waited on
    int nq = tid == 0 ? atomicAdd(a.work, 1) : 0;
    for (int k = 0; pos < count; ++k) {
        const int row = __ldg(a.rows + pos);
        if (tid == 0) {
            if (NB == 2) {
                bulk_wait_read0();  // the previous row's TMA store has finished reading its buffer
                issue_load(pos, buf, &bar[k & 1], k & 1);
            }
            np = nq;
            nq = atomicAdd(a.work, 1);  // consumed at the next row's start
            s_pos[2 + (k & 1)] = np;    // read at this row's end (visible after its first layer barrier)
            if (NB == 2 && np < count && a.l2_prefetch && !a.ybits)  // pull it into L2: its load is short
                bulk_prefetch_l2(a.yin + (size_t)__ldg(a.rows + np) * N, N * 4);
            if (NB == 3) {
                if (np < count) {  // load it now, behind this row's compute
                    // its buffer held the previous row's result: wait until that row's TMA store has read
                    // it (older stores were waited for one row earlier; constant-row stores read s_cz/s_cy)
                    if (prev_res) bulk_wait_read0();
                    issue_load(np, buf + i_pf * S, &bar[(k + 1) & 1], (k + 1) & 1);
                }
            }
        }
        mbar_wait(&bar[k & 1], (ph >> (k & 1)) & 1u);
        ph ^= 1u << (k & 1);
        // packed rows whose layer 0 runs as R32 are never expanded (layer 0 reads the bitmap only)
        if (a.ybits && !(a.popc0 && (p.L[0].flags & 15) == PF_NU1)) {  // expand the bits (value a.one) + halo
            float* dst = buf + i_in * S;
            const uint32_t* sb = s_bits + (k & 1) * (N / 32);
            const int wq = tid >> 5, lane = tid & 31;
#pragma unroll 4
            for (int j = 0; j < 32; ++j) {  // warp wq: words 32 wq .. 32 wq + 31, lane = bit (conflict-free)
                const int wi = wq * 32 + j;
                const float val = ((sb[wi] >> lane) & 1u) ? a.one : 0.0f;
                dst[wi * 32 + lane] = val;
                if (wi * 32 < H) dst[N + wi * 32 + lane] = val;
            }
            __syncthreads();
        }
        float* in = buf + i_in * S;
        float* out = buf + i_out * S;
        bool cst = false, dead = false;
        float v = 0.0f;
        int full = 0, full_fma = 0;  // layers evaluated in full; of them by fma chains (not R32)
        bool popc = false;
        bool r31_failed = false;  // R31 ran on this row without deciding it (R34 then runs at stride-1 layers)
        unsigned cmn = 0u, cmx = 0xffffffffu;  // the previous layer's output range (bits)
        int lend = a.t;  // the layer that zeroed the row (dead, R23), or t: alive after layer l <=> lend > l
        for (int l = 0; l < a.t; ++l) {
            // WUNI: one weight for every layer, read at a constant offset -> a uniform register operand
            const float w0 = WUNI ? p.L[0].w0 : p.L[l].w0, b0 = p.L[l].b0;
            const int fl = p.L[l].flags;
            const bool dead_next = (fl >> 4) & 1;
            if (!cst) {
                float mn = __int_as_float(0x7f800000), mx = -__int_as_float(0x7f800000);
                // range prediction (R30, exact; one weight w0 >= 0 and one bias for every layer < t): each
                // output is an fma chain + sigma, monotone in every input, so after k more layers every
                // element lies in [out^k(min), out^k(max)] of the previous layer's range.  min >= thr_hi[k-1]
                // with k = t - l: Y(t) is the constant row YMAX; max <= thr_lo[k-1]: Y(t) is zero (the row is
                // dropped at layer l - 1 + k, the layer by which it is proven zero).
                if (a.thr_ok && l > 0) {
                    const int rem = a.t - l;
                    const int kh = min(rem, kPfThr), kl = kh;
                    const float pmn = __uint_as_float(cmn), pmx = __uint_as_float(cmx);
                    if (pmn >= p.thr_hi[kh - 1]) {  // YMAX from layer l - 1 + kh on (a fixed point of the rest)
                        v = a.ymax;
                        cst = true;
                        break;
                    }
                    if (pmx <= p.thr_lo[kl - 1]) {  // zero from layer l - 1 + kl on (b0 <= 0: absorbing)
                        v = 0.0f;
                        cst = true;
                        if (a.drop && (kl == 1 ? dead_next : a.dead_t)) {
                            dead = true;
                            lend = l + kl - 1;
                            break;
                        }
                        if (kl == 1) continue;
                        break;
                    }
                }
                const int cls = fl & 15;
                // R32: layer 0 of stride 1 on a row of zeros and one value c.  fma(0, w0, acc) = acc exactly,
                // so every chain is k fmas of c from +0 (k = count of c in the window, in any order): the
                // output is tab[k], 33 values; the windows' counts are popcounts of the row's bitmap
                if (l == 0 && cls == PF_NU1 && (a.popc0 == 1 || (a.popc0 == 2 && a.ybits))) {
                    if (pf_popc_layer0<T>(in, out, a.ybits ? s_bits + (k & 1) * (N / 32) : nullptr, a.one, w0, b0,
                                          a.ymax, H, s_red, s_tabw, mn, mx)) {
                        popc = true;
                        goto layer_done;
                    }
                }
                // R31: a Q32 layer's outputs are bounded by its class sums (pf_q32_bounds) before they are
                // evaluated; R34: a stride-1 layer's by sliding window sums (pf_nu1_bounds; only after a
                // failed R31: the rows that reach such a layer late); the bounds of Y(l + 1) against the
                // horizon k = t - l - 1 decide as in R30
                if ((cls == PF_Q32 || (cls == PF_NU1 && a.win_bounds && r31_failed)) && a.thr_ok && l > 0) {
                    float ylo, yhi;
                    if (cls == PF_Q32) {
                        pf_q32_bounds<T>(in, w0, b0, a.ymax, ylo, yhi);
                        r31_failed = true;  // (if they decide the row it ends here)
                    } else {
                        pf_nu1_bounds<T>(in, w0, b0, a.ymax, ylo, yhi);
                    }
                    const unsigned wmn = __reduce_min_sync(0xffffffffu, __float_as_uint(ylo + 0.0f));
                    const unsigned wmx = __reduce_max_sync(0xffffffffu, __float_as_uint(yhi + 0.0f));
                    if ((tid & 31) == 0) {
                        s_bmn[tid >> 5] = wmn;
                        s_bmx[tid >> 5] = wmx;
                    }
                    __syncthreads();
                    const int ln = tid & 31;
                    const float bmn =
                        __uint_as_float(__reduce_min_sync(0xffffffffu, ln < kWarps ? s_bmn[ln] : 0xffffffffu));
                    const float bmx = __uint_as_float(__reduce_max_sync(0xffffffffu, ln < kWarps ? s_bmx[ln] : 0u));
                    const int k2 = a.t - l - 1;  // layers after this one
                    const int kk = min(k2, kPfThr);
                    if (bmn >= (k2 ? p.thr_hi[kk - 1] : a.ymax)) {  // Y(t) is the constant row YMAX
                        v = a.ymax;
                        cst = true;
                        break;
                    }
                    if (bmx <= (k2 ? p.thr_lo[kk - 1] : 0.0f)) {  // Y(t) is zero
                        v = 0.0f;
                        cst = true;
                        if (a.drop && (k2 ? a.dead_t : dead_next)) {
                            dead = true;
                            lend = l + kk;
                        }
                        break;
                    }
                }
                if (cls == PF_NU1)
                    pf_body_nu1<T>(in, out, w0, b0, a.ymax, H, mn, mx);
                else if (cls == PF_Q32)
                    pf_body_q32<T>(in, out, w0, b0, a.ymax, H, mn, mx);
                else if (GENSTR && p.L[l].nu != 32)
                    pf_body_str<T, 0, kPfStrHalo<T>>(in, out, p.L[l].nu, w0, b0, a.ymax, H, mn, mx);
                else
                    pf_body_str<T, 32, kPfStrHalo<T>>(in, out, 32, w0, b0, a.ymax, H, mn, mx);
                ++full_fma;
            layer_done:
                // the row's output range in one barrier: each warp publishes its (min, max) (bits of
                // outputs >= 0, -0 as +0, so bit order is value order and equal bits are equal values); after
                // the barrier every warp reduces the kWarps entries (slots double-buffered by layer parity)
                {
                    const unsigned wmn = __reduce_min_sync(0xffffffffu, __float_as_uint(mn + 0.0f));
                    const unsigned wmx = __reduce_max_sync(0xffffffffu, __float_as_uint(mx + 0.0f));
                    if ((tid & 31) == 0) {
                        s_vmn[(gl & 1) * kWarps + (tid >> 5)] = wmn;
                        s_vmx[(gl & 1) * kWarps + (tid >> 5)] = wmx;
                    }
                }
                __syncthreads();  // outputs and ranges written
                {
                    const int ln = tid & 31;
                    cmn = __reduce_min_sync(0xffffffffu, ln < kWarps ? s_vmn[(gl & 1) * kWarps + ln] : 0xffffffffu);
                    cmx = __reduce_max_sync(0xffffffffu, ln < kWarps ? s_vmx[(gl & 1) * kWarps + ln] : 0u);
                    ++gl;
                }
                const bool all_eq = cmn == cmx;  // every output equal (R26)
                const float o0 = __uint_as_float(cmn);
                ++full;
                float* tmp = in;
                in = out;
                out = tmp;
                const int ti = i_in;
                i_in = i_out;
                i_out = ti;
                if (all_eq) {
                    v = o0;
                    if (a.const_skip) cst = true;
                    if (v == 0.0f && a.drop && dead_next) {
                        dead = true;
                        lend = l;
                        break;
                    }
                }
            } else {
                // constant row (R26): v' = sigma(chain(v) + b0).  chain(+-0) = +0 exactly, and the host
                // evaluated chain(YMAX) with the same fma order (ymax_fixed)
                if (v == 0.0f) {
                    v = sigma(0.0f + b0, a.ymax);
                } else if (!(v == a.ymax && ((fl >> 5) & 1))) {
                    float acc = 0.0f;
#pragma unroll
                    for (int n = 0; n < 32; ++n) acc = fmaf(v, w0, acc);
                    v = sigma(acc + b0, a.ymax);
                }
                if (v == 0.0f && a.drop && dead_next) {
                    dead = true;
                    lend = l;
                    break;
                }
                // fixed point for every remaining layer: nothing more to evaluate (uncompressed path: t = L)
                if ((v == a.ymax && ((fl >> 6) & 1)) || (v == 0.0f && dead_next)) break;
            }
        }
        if (NB == 3 && tid == 0) prev_res = false;
        if (dead && a.ydead) {  // final activations of a dead row: zeros, written now (the SMs' HBM is idle)
            if (NB == 3) {  // one 4 KB bulk store per lane of warp 0 (issued in parallel, not by one thread)
                if (tid < N / kPfConstChunk) {
                    bulk_s2g(a.ydead + (size_t)row * N + tid * kPfConstChunk, s_cz, kPfConstChunk * 4);
                    bulk_commit();
                }
            } else {
                float4* dz = reinterpret_cast<float4*>(a.ydead + (size_t)row * N);
#pragma unroll
                for (int i = 0; i < N / 4 / T; ++i) dz[i * T + tid] = make_float4(0.f, 0.f, 0.f, 0.f);
            }
        }
        if (!dead) {
            float* gout = a.yout + (size_t)row * N;
            if (cst) {
                const uint32_t vb = __float_as_uint(v);
                if (NB == 3 && (vb == __float_as_uint(a.ymax) || vb == 0u)) {  // bitwise +0 / YMAX rows
                    if (tid < N / kPfConstChunk) {  // one 4 KB bulk store per lane of warp 0
                        bulk_s2g(gout + tid * kPfConstChunk, vb == 0u ? s_cz : s_cy, kPfConstChunk * 4);
                        bulk_commit();
                    }
                } else {
                    const float4 v4 = make_float4(v, v, v, v);
#pragma unroll
                    for (int i = 0; i < N / 4 / T; ++i) reinterpret_cast<float4*>(gout)[i * T + tid] = v4;
                }
            } else {
                fence_proxy_async_smem();  // generic-proxy writes of `in` -> visible to the TMA engine
                __syncthreads();
                if (tid == 0) {
                    bulk_s2g(gout, in, N * 4);
                    bulk_commit();
                    prev_res = true;
                }
            }
            if (tid == 0 && a.app_list) {
                s_surv[nsurv++] = row;
                flush_surv(false);
            }
            if (tid == 0 && a.rconst && cst) {  // constant at t: conversion needs no read of the row
                a.rconst[row] = 1;
                a.rval[row] = v;
            }
        }
        if (tid == 0) {
            if (a.full_rl) {
                atomicAdd(a.full_rl, (unsigned long long)full_fma);
                if (popc) atomicAdd(a.full_rl + 1, 1ull);
            }
            if (a.n_const && cst) atomicAdd(a.n_const, 1);
            if (a.dyn) {  // per-layer dynamics: histograms of the full-evaluation count and of the end layer
                atomicAdd(a.dyn + full, 1ull);
                atomicAdd(a.dyn + (a.t + 1) + lend, 1ull);
            }
        }
        pos = s_pos[2 + (k & 1)];
        if (NB == 3) {  // the prefetched row becomes the input; the result buffer (store pending) the target
            const int ti = i_in;
            i_in = i_pf;
            i_pf = ti;
        } else {
            i_in = 0;
            i_out = 1;
        }
    }
    if (a.app_list) flush_surv(true);
    if (tid < 32) bulk_wait0();  // every lane that issued bulk stores (constant rows: warp 0's lanes)
}

int pre_fused_threads(int N) {
    if (N % 32 != 0) return 0;
    const int T = N / 32;
    return (T == 32 || T == 64 || T == 128 || T == 256 || T == 512) ? T : 0;
}

size_t pre_fused_smem(int N, int H) {
    const int nb = N / 32 >= 512 ? 3 : 2;  // kPfBufs
    return sizeof(float) * nb * (size_t)(N + H) + 2 * sizeof(uint64_t) + 4 * sizeof(int) + 12 * sizeof(int) * (N / 32 / 32) +
           2 * sizeof(uint32_t) * (size_t)(N / 32) + sizeof(int) * kPfSurv +  // packed-row slots, survivors
           sizeof(float) * kPfTabStride * (N / 32 / 32) +                    // R32 tables
           (nb == 3 ? 2 * sizeof(float) * kPfConstChunk : 0);                 // constant-row store sources
}

template <int T, bool GENSTR, bool WUNI>
static cudaError_t launch_tg(const PreFusedParams& p, int num_sms, cudaStream_t st) {
    const size_t smem = pre_fused_smem(p.a.N, p.a.H);
    int bps = 0;
    cudaError_t e = blocks_per_sm((const void*)pre_fused_kernel<T, GENSTR, WUNI>, T, smem, &bps);
    if (e != cudaSuccess) return e;
    if (bps < 1) return cudaErrorInvalidConfiguration;
    pre_fused_kernel<T, GENSTR, WUNI><<<num_sms * bps, T, smem, st>>>(p);
    return cudaGetLastError();
}
template <int T>
static cudaError_t launch_t(const PreFusedParams& p, bool wuni, int num_sms, cudaStream_t st) {
    if (p.a.gen_str) return wuni ? launch_tg<T, true, true>(p, num_sms, st) : launch_tg<T, true, false>(p, num_sms, st);
    return wuni ? launch_tg<T, false, true>(p, num_sms, st) : launch_tg<T, false, false>(p, num_sms, st);
}

cudaError_t launch_pre_fused(const PreFusedArgs& a, const PreFusedLayer* layers, int num_sms, cudaStream_t st) {
    if (a.t < 1 || a.t > kPfMaxLayers) return cudaErrorInvalidValue;
    static thread_local PreFusedParams p;  // 32 KB: not on the stack
    p.a = a;
    p.a.l2_prefetch = 1;  // measured neutral on C2 (row loads are short anyway); kept for larger rows
    for (int l = 0; l < a.t; ++l) {
        p.L[l].w0 = layers[l].w0;
        p.L[l].b0 = layers[l].b0;
        p.L[l].nu = layers[l].nu;
        p.L[l].flags = (layers[l].cls & 15) | (layers[l].dead_next ? 16 : 0) | (layers[l].ymax_fixed ? 32 : 0);
    }
    // bit 6: YMAX is a fixed point of every layer l + 1 .. t-1 (a constant YMAX row after layer l needs
    // no more evaluation)
    for (int l = a.t - 1, all = 1; l >= 0; --l) {
        if (all) p.L[l].flags |= 64;
        all = all && layers[l].ymax_fixed;
    }
    // range prediction horizon tables (R30, kernels_const.cu)
    p.a.thr_ok = a.const_skip && a.range_pred && range_tables(layers, a.t, a.ymax, p.thr_hi, p.thr_lo);
    p.a.dead_t = layers[a.t - 1].dead_next;
    bool wuni = true;
    for (int l = 1; l < a.t; ++l) wuni = wuni && memcmp(&p.L[l].w0, &p.L[0].w0, sizeof(float)) == 0;
    switch (pre_fused_threads(a.N)) {
        case 32: return launch_t<32>(p, wuni, num_sms, st);
        case 64: return launch_t<64>(p, wuni, num_sms, st);
        case 128: return launch_t<128>(p, wuni, num_sms, st);
        case 256: return launch_t<256>(p, wuni, num_sms, st);
        case 512: return launch_t<512>(p, wuni, num_sms, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace snicit
