// kernels_pre_cluster.cu -- row-resident pre-convergence phase (a1) for large rows, sm_100a.
//
// Same computation as kernels_pre_fused.cu (Eq. 1, layers 0..t-1 of a row kept on chip, the
// stored-order fma chains of R12 with packed FFMA2, constant rows R26, dead rows R23), for rows that a
// single CTA can only hold at one CTA per SM (N = 16384: 64 KB rows, 512 threads, 86 registers) or not at
// all (N = 65536: 256 KB rows).  A row is split over a thread-block cluster of G = N / 8192 CTAs: every
// CTA owns S = 8192 outputs per layer (256 threads x 32 outputs), keeps only its share of the row (two
// buffers of S + halo floats, 74 KB) and runs at three CTAs per SM, so the layer barriers of one row are
// covered by the other rows' work (one CTA per SM left the FMA pipe idle during every layer's
// load / epilogue phase: 60% of its peak at N = 16384).
//
// Partitions (chosen per layer by its stride class so that each CTA's inputs are a compact local set):
//   W  (nu == 1, and strided layers with Q/G >= 32 a-rows per CTA): CTA r owns outputs
//      [r S, (r + 1) S); its buffer holds y[(r S + x) mod N], x < S + Hh (window + circular halo).
//   C  (Q = N/nu < 32 G: the Q == 32 class, and Q = 64 / 128 strided layers): CTA r owns residue
//      classes c in [r nu/G, (r + 1) nu/G) at every a-row; its buffer holds y[a nu + r nu/G + c'] at
//      a (nu/G) + c'.
// Every output is stored straight into the buffer of the CTA that owns it under the NEXT layer's
// partition (and into a second CTA's halo when it lies in one), through distributed shared memory
// (st.shared::cluster); one cluster barrier per layer orders the exchange.  The arithmetic of every
// output is exactly that of kernels_pre_fused.cu, so results are bit-identical (tested).
#include <cuda_runtime.h>

#include <cstring>

#include "snicit_internal.cuh"

namespace snicit {

constexpr int kCS = 8192;       // outputs per CTA per layer
constexpr int kCLS = 13;        // log2(kCS)
constexpr int kCT = kCS / 32;   // threads per CTA
constexpr int kCWp = kCT / 32;  // warps per CTA
constexpr int kCSurv = 32;
#ifndef SNICIT_CF_MINBLOCKS
#define SNICIT_CF_MINBLOCKS 3
#endif
constexpr int kCfMinBlocks = SNICIT_CF_MINBLOCKS;  // CTAs per SM the register budget is sized for

typedef unsigned long long u64;

enum CfClass : int { CF_NU1 = 0, CF_WSTR = 1, CF_CSTR = 2, CF_Q32 = 3 };

struct CfLayer {
    float w0, b0;
    int nu;
    int flags;  // cls | dead_next << 4 | ymax_fixed << 5
};
constexpr int kCfMaxLayers = kPfMaxLayers - 20;  // (parameter space: the R30 tables below)
struct CfParams {
    PreFusedArgs a;
    int Hh;        // W-partition halo (floats)
    int pad;
    float thr_hi[kRangeK], thr_lo[kRangeK];  // R30 horizon tables (kernels_const.cu range_tables)
    CfLayer L[kCfMaxLayers + 1];  // L[t]: sentinel (the output of layer t-1 is stored in the W partition)
};
static_assert(sizeof(CfParams) <= 32764, "kernel parameter space");

__device__ __forceinline__ uint32_t mapa_u32(uint32_t a, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(rank));
    return r;
}
__device__ __forceinline__ void st_cl_f32(uint32_t addr, float v) {
    asm volatile("st.shared::cluster.f32 [%0], %1;" ::"r"(addr), "f"(v) : "memory");
}
__device__ __forceinline__ void st_cl_u32(uint32_t addr, uint32_t v) {
    asm volatile("st.shared::cluster.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}
__device__ __forceinline__ void cluster_barrier() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t cluster_ctarank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ int ilog2i(int x) { return 31 - __clz(x); }

// Where output q (global index) goes under the next layer's partition: one or two (rank, offset) slots.
// RT_LOC: this layer and the next are both W-partitioned -- the output is this CTA's own (local offset
// q - q0), plus a copy into the previous rank's halo for the first Hh outputs; RT_W: next layer W, this
// one C; RT_C: next layer C (residue partition of nu').  The mode is a template parameter of the bodies
// so each instantiation has one straight store path.
enum RouteMode : int { RT_LOC = 0, RT_W = 1, RT_C = 2 };
struct Router {
    int hh;      // W halo
    int lnu;     // C: log2(nu'), log2(nu'/G)
    int lnug;
    int gmask;   // G - 1
    int q0;      // r S
    float* outl;          // local next-layer buffer
    uint32_t halo_base;   // cluster address of the previous rank's next-layer buffer + 4 S
    const uint32_t* base;  // [G] cluster addresses of the next-layer buffer of each rank
    template <int MODE>
    __device__ __forceinline__ void put(int q, float v) const {
        if constexpr (MODE == RT_LOC) {
            const int off = q - q0;
            outl[off] = v;
            if (off < hh) st_cl_f32(halo_base + 4u * (uint32_t)off, v);
        } else if constexpr (MODE == RT_W) {
            const int h = q >> kCLS, off = q & (kCS - 1);
            st_cl_f32(base[h] + 4u * (uint32_t)off, v);
            if (off < hh) st_cl_f32(base[(h - 1) & gmask] + 4u * (uint32_t)(kCS + off), v);
        } else {
            const int a = q >> lnu, c = q & ((1 << lnu) - 1);
            const int h = c >> lnug;
            const int off = (a << lnug) | (c & ((1 << lnug) - 1));
            st_cl_f32(base[h] + 4u * (uint32_t)off, v);
        }
    }
};

// ---------------------------------------------------------------------------- layer bodies (one CTA's share)
// W, nu == 1: local outputs [17i, 17i + 17) and [17T + 15i, 17T + 15i + 15) of the CTA's window
// (exact tiling of S = 32T, odd lane strides: conflict-free LDS); 15 FFMA2 pairs + 2 scalar chains.
template <int MODE>
__device__ __forceinline__ void cf_body_nu1(const float* __restrict__ in, int q0, float w0, float b0, float ymax,
                                            const Router& rt, float& mn, float& mx) {
    constexpr int T = kCT;
    constexpr int M1 = 17, M2 = 15, W2N = M2 + 31;
    const int i1 = threadIdx.x;
    const float* s1 = in + M1 * i1;
    const float* s2 = in + M1 * T + M2 * i1;
    u64 R[W2N];
#pragma unroll
    for (int i = 0; i < W2N; ++i) R[i] = f2_pack(s1[i], s2[i]);
    const float e46 = s1[W2N], e47 = s1[W2N + 1];
    const u64 W2 = f2_pack(w0, w0), B2 = f2_pack(b0, b0);
    const int qa = q0 + M1 * i1, qb = q0 + M1 * T + M2 * i1;
#pragma unroll
    for (int m = 0; m < M2; ++m) {
        u64 acc = 0ull;
#pragma unroll
        for (int n = 0; n < 32; ++n) acc = f2_fma(R[m + n], W2, acc);
        float z1, z2;
        f2_unpack(f2_add(acc, B2), z1, z2);
        const float o1 = sigma(z1, ymax), o2 = sigma(z2, ymax);
        rt.template put<MODE>(qa + m, o1);
        rt.template put<MODE>(qb + m, o2);
        mn = fminf(mn, fminf(o1, o2));
        mx = fmaxf(mx, fmaxf(o1, o2));
    }
#pragma unroll
    for (int m = M2; m < M1; ++m) {
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
        rt.template put<MODE>(qa + m, o1);
        mn = fminf(mn, o1);
        mx = fmaxf(mx, o1);
    }
}

// W, strided (nu >= 32, Q/G >= 32 a-rows per CTA): item (c, a0) = local outputs (a0 + m) nu + c,
// m < 16, paired with (c, a0 + P), P = Q/(2G) -- both inside the CTA's a-range; lanes on consecutive c.
template <int NU, int MODE>
__device__ __forceinline__ void cf_body_wstr(const float* __restrict__ in, int q0, int nu_rt, int P, float w0,
                                             float b0, float ymax, const Router& rt, float& mn, float& mx) {
    const int nu = NU ? NU : nu_rt;
    const int c = (int)threadIdx.x % nu;
    const int a0 = ((int)threadIdx.x / nu) * 16;
    const int base = a0 * nu + c;
    const int off2 = P * nu;
    const float* s = in + base;
    u64 R[47];
#pragma unroll
    for (int i = 0; i < 47; ++i) R[i] = f2_pack(s[i * nu], s[i * nu + off2]);
    const u64 W2 = f2_pack(w0, w0), B2 = f2_pack(b0, b0);
#pragma unroll
    for (int m = 0; m < 16; ++m) {
        u64 acc = 0ull;
#pragma unroll
        for (int n = 0; n < 32; ++n) acc = f2_fma(R[m + n], W2, acc);
        float z1, z2;
        f2_unpack(f2_add(acc, B2), z1, z2);
        const float o1 = sigma(z1, ymax), o2 = sigma(z2, ymax);
        const int q1 = q0 + base + m * nu;
        rt.template put<MODE>(q1, o1);
        rt.template put<MODE>(q1 + off2, o2);
        mn = fminf(mn, fminf(o1, o2));
        mx = fmaxf(mx, fmaxf(o1, o2));
    }
}

// C, strided with few a-rows (Q = 64 / 128): residue c' of the CTA's nu/G classes, a-block a0 in
// {0, 16, ..} < Q/2, paired with a0 + Q/2; a-row indices wrap mod Q (power of two).
template <int MODE>
__device__ __forceinline__ void cf_body_cstr(const float* __restrict__ in, int r, int nu, int Q, float w0, float b0,
                                             float ymax, const Router& rt, float& mn, float& mx, int lnug) {
    const int nug = 1 << lnug;
    const int cp = (int)threadIdx.x & (nug - 1);
    const int a0 = ((int)threadIdx.x >> lnug) * 16;
    const int h2 = Q / 2;
    const float* sc = in + cp;
    u64 R[47];
#pragma unroll
    for (int i = 0; i < 47; ++i)
        R[i] = f2_pack(sc[((a0 + i) & (Q - 1)) << lnug], sc[((a0 + h2 + i) & (Q - 1)) << lnug]);
    const u64 W2 = f2_pack(w0, w0), B2 = f2_pack(b0, b0);
    const int cg = r * nug + cp;
#pragma unroll
    for (int m = 0; m < 16; ++m) {
        u64 acc = 0ull;
#pragma unroll
        for (int n = 0; n < 32; ++n) acc = f2_fma(R[m + n], W2, acc);
        float z1, z2;
        f2_unpack(f2_add(acc, B2), z1, z2);
        const float o1 = sigma(z1, ymax), o2 = sigma(z2, ymax);
        rt.template put<MODE>((a0 + m) * nu + cg, o1);
        rt.template put<MODE>((a0 + h2 + m) * nu + cg, o2);
        mn = fminf(mn, fminf(o1, o2));
        mx = fmaxf(mx, fmaxf(o1, o2));
    }
}

// C, Q == 32 (nu = N/32): thread c' owns residue class r T + c' -- its 32 inputs are local; items a0 = 0
// and a0 = 16; every rotation compile-time.
template <int NU, int MODE>
__device__ __forceinline__ void cf_body_q32(const float* __restrict__ in, int r, float w0, float b0, float ymax,
                                            const Router& rt, float& mn, float& mx) {
    constexpr int T = kCT;
    const int cp = threadIdx.x;
    float x[32];
#pragma unroll
    for (int k = 0; k < 32; ++k) x[k] = in[k * T + cp];
    u64 P[32];
#pragma unroll
    for (int k = 0; k < 32; ++k) P[k] = f2_pack(x[k], x[(k + 16) & 31]);
    const u64 W2 = f2_pack(w0, w0), B2 = f2_pack(b0, b0);
    const int cg = r * T + cp;
#pragma unroll
    for (int m = 0; m < 16; ++m) {
        u64 acc = 0ull;
#pragma unroll
        for (int n = 0; n < 32; ++n) acc = f2_fma(P[(m + n) & 31], W2, acc);
        float z1, z2;
        f2_unpack(f2_add(acc, B2), z1, z2);
        const float o1 = sigma(z1, ymax), o2 = sigma(z2, ymax);
        rt.template put<MODE>(m * NU + cg, o1);
        rt.template put<MODE>((m + 16) * NU + cg, o2);
        mn = fminf(mn, fminf(o1, o2));
        mx = fmaxf(mx, fmaxf(o1, o2));
    }
}

// ---------------------------------------------------------------------------- specialised routes
// The transitions of the SDGC stride cycles (N = 16384: nu 1 -> 32 -> 512 -> 1; N = 65536: 1 -> 32 ->
// 1024 -> 2048 -> 1) with the routing folded into per-thread base addresses and compile-time offsets:
// for output m of an item the target rank and offset are affine in m (derivations at each body), so a
// store costs one st.shared::cluster with an immediate offset instead of the generic Router's integer work
// (measured: the generic routing made the kernel issue-bound, 45% more instructions).

// W, nu = 32 -> C(NNU) (NNU >= 512, nu'/G = NNU/G in [32, 512]).  Item base Qi = Qhi + c with Qhi a
// multiple of 512 (q0 = r S, a0 32 with a0 a multiple of 16) and c < 32, so with b = Qhi mod NNU (a
// multiple of 512, hence of nu'/G): output Qi + 32 m (m < 16) has residue b + c + 32 m, owner rank
// (b >> lnug) + (32 m >> lnug) and offset ((Qhi >> lnu) << lnug) + c + (32 m & (nu'/G - 1)).
template <int G, int NNU>
__device__ __forceinline__ void sp_wstr32_c(const float* __restrict__ in, int q0, float w0, float b0, float ymax,
                                            const uint32_t* nb, float& mn, float& mx) {
    constexpr int NUG = NNU / G;
    constexpr int LNU = __builtin_ctz(NNU), LNUG = __builtin_ctz(NUG);
    constexpr int NB = (16 * 32 + NUG - 1) / NUG;  // ranks one item's 16 outputs span
    constexpr int P32 = (kCS / 2);                 // second item: + P nu = S / 2
    const int c = (int)threadIdx.x & 31;
    const int a0 = ((int)threadIdx.x >> 5) * 16;
    const float* s = in + a0 * 32 + c;
    u64 R[47];
#pragma unroll
    for (int i = 0; i < 47; ++i) R[i] = f2_pack(s[i * 32], s[i * 32 + P32]);
    uint32_t B1[NB], B2[NB];
    {
        const int Qhi1 = q0 + a0 * 32, Qhi2 = Qhi1 + P32;
        const int hb1 = (Qhi1 & (NNU - 1)) >> LNUG, hb2 = (Qhi2 & (NNU - 1)) >> LNUG;
        const uint32_t o1 = 4u * (uint32_t)(((Qhi1 >> LNU) << LNUG) + c), o2 = 4u * (uint32_t)(((Qhi2 >> LNU) << LNUG) + c);
#pragma unroll
        for (int k = 0; k < NB; ++k) {
            B1[k] = nb[hb1 + k] + o1;
            B2[k] = nb[hb2 + k] + o2;
        }
    }
    const u64 W2 = f2_pack(w0, w0), BB = f2_pack(b0, b0);
#pragma unroll
    for (int m = 0; m < 16; ++m) {
        u64 acc = 0ull;
#pragma unroll
        for (int n = 0; n < 32; ++n) acc = f2_fma(R[m + n], W2, acc);
        float z1, z2;
        f2_unpack(f2_add(acc, BB), z1, z2);
        const float o1 = sigma(z1, ymax), o2 = sigma(z2, ymax);
        st_cl_f32(B1[(32 * m) >> LNUG] + 4u * (uint32_t)((32 * m) & (NUG - 1)), o1);
        st_cl_f32(B2[(32 * m) >> LNUG] + 4u * (uint32_t)((32 * m) & (NUG - 1)), o2);
        mn = fminf(mn, fminf(o1, o2));
        mx = fmaxf(mx, fmaxf(o1, o2));
    }
}

// C, Q = 32 (nu = N/32, a multiple of S / 32 ... S is a multiple of nu) -> W.  Output m nu + cg (cg =
// r nu/G + c' < nu): owner rank (m nu) >> 13, offset (m nu mod S) + cg; halo copy when that offset < Hh.
template <int N>
__device__ __forceinline__ void sp_q32_w(const float* __restrict__ in, int r, float w0, float b0, float ymax, int hh,
                                         const uint32_t* nb, float& mn, float& mx) {
    constexpr int G = N / kCS, NU = N / 32, T = kCT;
    const int cp = threadIdx.x;
    float x[32];
#pragma unroll
    for (int k = 0; k < 32; ++k) x[k] = in[k * T + cp];
    u64 P[32];
#pragma unroll
    for (int k = 0; k < 32; ++k) P[k] = f2_pack(x[k], x[(k + 16) & 31]);
    const u64 W2 = f2_pack(w0, w0), BB = f2_pack(b0, b0);
    const int cg = r * T + cp;
    const uint32_t o = 4u * (uint32_t)cg;
#pragma unroll
    for (int m = 0; m < 16; ++m) {
        u64 acc = 0ull;
#pragma unroll
        for (int n = 0; n < 32; ++n) acc = f2_fma(P[(m + n) & 31], W2, acc);
        float z1, z2;
        f2_unpack(f2_add(acc, BB), z1, z2);
        const float o1 = sigma(z1, ymax), o2 = sigma(z2, ymax);
#pragma unroll
        for (int it = 0; it < 2; ++it) {
            const int mm = m + 16 * it;
            const int h = (mm * NU) >> kCLS, off0 = (mm * NU) & (kCS - 1);  // compile-time
            const float v = it ? o2 : o1;
            st_cl_f32(nb[h] + o + 4u * (uint32_t)off0, v);
            if (off0 < 1024 && off0 + cg < hh)  // the previous rank's halo
                st_cl_f32(nb[(h - 1) & (G - 1)] + o + 4u * (uint32_t)(kCS + off0), v);
        }
        mn = fminf(mn, fminf(o1, o2));
        mx = fmaxf(mx, fmaxf(o1, o2));
    }
}

// C, Q = 64 (nu = N/64) -> C(2 nu).  Output (a + m) nu + cg (a in {a0, a0 + 32}, a0 in {0, 16}, cg = r nu/G + c'):
// residue of 2 nu is (m & 1) nu + cg, so with nu'/G = 2 nu / G the owner rank is (m & 1) (nu >> lnug') +
// (cg >> lnug') and the offset (((a >> 1) + (m >> 1)) << lnug') + (cg & (nu'/G - 1)).
template <int N>
__device__ __forceinline__ void sp_cstr_c2(const float* __restrict__ in, int r, float w0, float b0, float ymax,
                                           const uint32_t* nb, float& mn, float& mx) {
    constexpr int G = N / kCS, NU = N / 64, Q = 64;
    constexpr int NUG = NU / G, LNUG = __builtin_ctz(NUG);
    constexpr int NUG2 = 2 * NU / G, LNUG2 = __builtin_ctz(NUG2);
    const int cp = (int)threadIdx.x & (NUG - 1);
    const int a0 = ((int)threadIdx.x >> LNUG) * 16;
    const float* sc = in + cp;
    u64 R[47];
#pragma unroll
    for (int i = 0; i < 47; ++i) R[i] = f2_pack(sc[((a0 + i) & (Q - 1)) * NUG], sc[((a0 + 32 + i) & (Q - 1)) * NUG]);
    const int cg = r * NUG + cp;
    uint32_t B1[2], B2[2];
#pragma unroll
    for (int k = 0; k < 2; ++k) {
        const uint32_t nbk = nb[k * (NU >> LNUG2) + (cg >> LNUG2)];
        B1[k] = nbk + 4u * (uint32_t)(((a0 >> 1) << LNUG2) + (cg & (NUG2 - 1)));
        B2[k] = nbk + 4u * (uint32_t)((((a0 + 32) >> 1) << LNUG2) + (cg & (NUG2 - 1)));
    }
    const u64 W2 = f2_pack(w0, w0), BB = f2_pack(b0, b0);
#pragma unroll
    for (int m = 0; m < 16; ++m) {
        u64 acc = 0ull;
#pragma unroll
        for (int n = 0; n < 32; ++n) acc = f2_fma(R[m + n], W2, acc);
        float z1, z2;
        f2_unpack(f2_add(acc, BB), z1, z2);
        const float o1 = sigma(z1, ymax), o2 = sigma(z2, ymax);
        st_cl_f32(B1[m & 1] + 4u * (uint32_t)((m >> 1) << LNUG2), o1);
        st_cl_f32(B2[m & 1] + 4u * (uint32_t)((m >> 1) << LNUG2), o2);
        mn = fminf(mn, fminf(o1, o2));
        mx = fmaxf(mx, fmaxf(o1, o2));
    }
}

// ---------------------------------------------------------------------------- the kernel
// G = N / kCS CTAs per cluster (launched with the cluster dimension set at launch); WUNI: one weight for
// every layer (read at a constant offset -> uniform-register FFMA2 operand).
template <int N, bool WUNI>
__global__ void __launch_bounds__(kCT, kCfMinBlocks) pre_cluster_kernel(const __grid_constant__ CfParams p) {
    constexpr int G = N / kCS;
    constexpr int T = kCT;
    constexpr int NU_Q32 = N / 32;
    const PreFusedArgs& a = p.a;
    const int Hh = p.Hh;
    const int BS = kCS + Hh;  // buffer stride (floats)
    extern __shared__ __align__(128) unsigned char smem[];
    float* const buf = reinterpret_cast<float*>(smem);               // [2][BS] (BS: multiple of 128)
    uint64_t* bar = reinterpret_cast<uint64_t*>(buf + 2 * BS);          // [2] row loads
    uint32_t* s_bits = reinterpret_cast<uint32_t*>(bar + 2);            // [(kCS + 1024) / 32] packed row (16 B aligned)
    int* s_pos = reinterpret_cast<int*>(s_bits + (kCS + 1024) / 32);    // [2] row position by row parity
    unsigned* s_vmn = reinterpret_cast<unsigned*>(s_pos + 2);           // [2][G * kCWp] warp output minima (bits)
    unsigned* s_vmx = s_vmn + 2 * G * kCWp;                             // [2][G * kCWp] warp output maxima
    uint32_t* s_base = reinterpret_cast<uint32_t*>(s_vmx + 2 * G * kCWp);  // [2][G] buffer b of rank h
    int* s_surv = reinterpret_cast<int*>(s_base + 2 * G);               // [kCSurv]
    unsigned* s_bmn = reinterpret_cast<unsigned*>(s_surv + kCSurv);      // [G * kCWp] Q32 class-sum bounds (R31)
    unsigned* s_bmx = s_bmn + G * kCWp;
    const int tid = threadIdx.x;
    const int r = (int)cluster_ctarank();
    const int count = *a.count;
    if (tid < 2 * G) {
        const int b = tid / G, h = tid % G;
        s_base[b * G + h] = mapa_u32(smem_u32(buf + b * BS), (uint32_t)h);
    }
    if (tid == 0) {
        mbar_init(&bar[0], 1);
        mbar_init(&bar[1], 1);
        fence_proxy_async_smem();
    }
    // every CTA of the cluster has started (and initialised its shared memory) before any remote access
    cluster_barrier();
    // the first row: rank 0 claims it for the cluster
    if (r == 0 && tid == 0) {
        const int p0 = atomicAdd(a.work, 1);
        for (int h = 0; h < G; ++h) st_cl_u32(mapa_u32(smem_u32(s_pos), (uint32_t)h), (uint32_t)p0);
    }
    cluster_barrier();
    int pos = s_pos[0];
    int nsurv = 0;
    // the first layer's partition decides how a row is loaded
    const int cls0 = p.L[0].flags & 15;
    const bool w0part = cls0 == CF_NU1 || cls0 == CF_WSTR;
    auto issue_load = [&](int p_, uint64_t* b) {
        const size_t r_ = (size_t)__ldg(a.rows + p_);
        if (a.ready) {  // streamed upload: wait for this row's chunk (geometric chunks, see launch)
            const int* f = a.ready + (31 - __clz((int)(r_ / a.ready_rows) + 1));
            while (ld_acquire_gpu(f) == 0) __nanosleep(256);
            fence_proxy_async_global();
        }
        if (a.ybits) {  // W partition only (checked by the host): the window's words + the halo's words
            const uint32_t* gb = a.ybits + r_ * (N / 32);
            mbar_arrive_expect_tx(b, (uint32_t)((kCS + Hh) / 8));
            bulk_g2s(s_bits, gb + r * (kCS / 32), kCS / 8, b);
            bulk_g2s(s_bits + kCS / 32, gb + (((r + 1) % G) * kCS) / 32, Hh / 8, b);
        } else if (w0part) {
            const float* g = a.yin + r_ * N;
            mbar_arrive_expect_tx(b, (uint32_t)(BS * 4));
            bulk_g2s(buf, g + (size_t)r * kCS, kCS * 4, b);
            bulk_g2s(buf + kCS, g + (size_t)((r + 1) % G) * kCS, Hh * 4, b);
        } else {  // C partition: Q a-rows of nu/G floats
            const float* g = a.yin + r_ * N;
            const int nu = p.L[0].nu, nug = nu / G, Q = N / nu;
            mbar_arrive_expect_tx(b, (uint32_t)(kCS * 4));
            for (int aa = 0; aa < Q; ++aa) bulk_g2s(buf + aa * nug, g + (size_t)aa * nu + (size_t)r * nug, nug * 4, b);
        }
    };
    uint32_t ph = 0;
    // The row-end cluster barrier is needed only when the next row's layer 0 writes into peers' row areas:
    // when layers 0 and 1 are both W-partitioned (the SDGC cycles), layer 0 writes remote HALOS only, which
    // no rank reads while it finishes a row (its result store reads [0, kCS)), so a rank may start the next
    // row at once (round 2 (r02c)).  Votes use a running layer-instance parity (gl) so the slots of a row's
    // last layer and the next row's first layer differ; a rank is never more than one row ahead of a peer
    // (it cannot pass the next row's layer-0 barrier alone).
    const int cls1 = a.t > 1 ? (p.L[1].flags & 15) : CF_NU1;
    const bool end_barrier = !(w0part && (cls1 == CF_NU1 || cls1 == CF_WSTR));
    int gl = 0;  // evaluated layer instances (vote slot parity)
    for (int k = 0; pos < count; ++k) {
        const int row = __ldg(a.rows + pos);
        if (tid == 0) issue_load(pos, &bar[0]);
        if (r == 0 && tid == 0) {  // next row for the cluster, visible after this row's first cluster barrier
            const int np = atomicAdd(a.work, 1);
            for (int h = 0; h < G; ++h)
                st_cl_u32(mapa_u32(smem_u32(s_pos + ((k + 1) & 1)), (uint32_t)h), (uint32_t)np);
        }
        mbar_wait(&bar[0], ph & 1u);
        ph ^= 1u;
        if (a.ybits) {  // expand the staged bits into buffer 0 (value a.one)
            for (int x = tid; x < kCS + Hh; x += T) buf[x] = ((s_bits[x >> 5] >> (x & 31)) & 1u) ? a.one : 0.0f;
            __syncthreads();
        }
        bool cst = false, dead = false;
        float v = 0.0f;
        int full = 0;
        int cur = 0;  // buffer holding this layer's input
        for (int l = 0; l < a.t; ++l) {
            const float w0 = WUNI ? p.L[0].w0 : p.L[l].w0, b0 = p.L[l].b0;
            const int fl = p.L[l].flags;
            const bool dead_next = (fl >> 4) & 1;
            if (!cst) {
                const float* in = buf + cur * BS;
                // router into the next layer's partition (layer t: W)
                Router rt;
                const int ncls = p.L[l + 1].flags & 15;
                const bool nw = (l + 1 >= a.t) || ncls == CF_NU1 || ncls == CF_WSTR;
                rt.hh = Hh;
                rt.gmask = G - 1;
                rt.q0 = r * kCS;
                rt.outl = buf + (cur ^ 1) * BS;
                rt.base = s_base + (cur ^ 1) * G;
                rt.halo_base = s_base[(cur ^ 1) * G + ((r - 1) & (G - 1))] + 4u * kCS;
                if (!nw) {
                    rt.lnu = ilog2i(p.L[l + 1].nu);
                    rt.lnug = rt.lnu - ilog2i(G);
                }
                float mn = __int_as_float(0x7f800000), mx = -__int_as_float(0x7f800000);
                const int cls = fl & 15;
                const int nu = p.L[l].nu;
                // R31 (kernels_pre_fused.cu pf_q32_bounds): in the C partition of a Q32 layer thread c owns
                // residue class r T + c, whose 32 outputs all sum its 32 inputs (buffer a T + c); directed-
                // rounding chains bound every output before any is evaluated, one extra cluster barrier
                // gathers the bounds, and the horizon k = t - l - 1 decides as in R30
                if (cls == CF_Q32 && a.thr_ok && l > 0 && NU_Q32 / G == T) {
                    float slo = 0.0f, shi = 0.0f;
#pragma unroll 8
                    for (int kq = 0; kq < 32; ++kq) {
                        const float x = in[kq * T + tid];
                        slo = __fmaf_rd(x, w0, slo);
                        shi = __fmaf_ru(x, w0, shi);
                    }
                    const float blo = __fsub_rd(__fmul_rd(slo, 1.0f - 0x1p-19f), 0x1p-140f);
                    const float bhi = __fadd_ru(__fmul_ru(shi, 1.0f + 0x1p-18f), 0x1p-140f);
                    const float ylo = sigma(__fadd_rd(blo, b0), a.ymax), yhi = sigma(__fadd_ru(bhi, b0), a.ymax);
                    const unsigned wmn = __reduce_min_sync(0xffffffffu, __float_as_uint(ylo + 0.0f));
                    const unsigned wmx = __reduce_max_sync(0xffffffffu, __float_as_uint(yhi + 0.0f));
                    if ((tid & 31) == 0) {
                        const int slot = r * kCWp + (tid >> 5);
                        for (int h = 0; h < G; ++h) {
                            st_cl_u32(mapa_u32(smem_u32(s_bmn + slot), (uint32_t)h), wmn);
                            st_cl_u32(mapa_u32(smem_u32(s_bmx + slot), (uint32_t)h), wmx);
                        }
                    }
                    cluster_barrier();
                    unsigned m0 = 0xffffffffu, m1 = 0u;
                    for (int w = tid & 31; w < G * kCWp; w += 32) {
                        m0 = min(m0, s_bmn[w]);
                        m1 = max(m1, s_bmx[w]);
                    }
                    const float bmn = __uint_as_float(__reduce_min_sync(0xffffffffu, m0));
                    const float bmx = __uint_as_float(__reduce_max_sync(0xffffffffu, m1));
                    const int k2 = a.t - l - 1;
                    const int kk = min(k2, kRangeK);
                    if (bmn >= (k2 ? p.thr_hi[kk - 1] : a.ymax)) {  // Y(t) is the constant row YMAX
                        v = a.ymax;
                        cst = true;
                        break;
                    }
                    if (bmx <= (k2 ? p.thr_lo[kk - 1] : 0.0f)) {  // Y(t) is zero
                        v = 0.0f;
                        cst = true;
                        if (a.drop && (k2 ? a.dead_t : dead_next)) dead = true;
                        break;
                    }
                }
                if (cls == CF_NU1) {
                    if (nw)
                        cf_body_nu1<RT_LOC>(in, r * kCS, w0, b0, a.ymax, rt, mn, mx);
                    else
                        cf_body_nu1<RT_C>(in, r * kCS, w0, b0, a.ymax, rt, mn, mx);
                } else if (cls == CF_WSTR) {
                    const int P = (N / nu) / (2 * G);
                    const int nnu = p.L[l + 1].nu;
                    if (nu == 32) {
                        if (nw)
                            cf_body_wstr<32, RT_LOC>(in, r * kCS, 32, P, w0, b0, a.ymax, rt, mn, mx);
                        else if (nnu == N / 32 && N / 32 / G >= 32 && N / 32 / G <= 512)
                            sp_wstr32_c<G, N / 32>(in, r * kCS, w0, b0, a.ymax, rt.base, mn, mx);
                        else if (nnu == N / 64 && N / 64 / G >= 32 && N / 64 / G <= 512)
                            sp_wstr32_c<G, N / 64>(in, r * kCS, w0, b0, a.ymax, rt.base, mn, mx);
                        else
                            cf_body_wstr<32, RT_C>(in, r * kCS, 32, P, w0, b0, a.ymax, rt, mn, mx);
                    } else {
                        if (nw)
                            cf_body_wstr<0, RT_LOC>(in, r * kCS, nu, P, w0, b0, a.ymax, rt, mn, mx);
                        else
                            cf_body_wstr<0, RT_C>(in, r * kCS, nu, P, w0, b0, a.ymax, rt, mn, mx);
                    }
                } else if (cls == CF_Q32) {
                    if (nw)
                        sp_q32_w<N>(in, r, w0, b0, a.ymax, Hh, rt.base, mn, mx);
                    else
                        cf_body_q32<NU_Q32, RT_C>(in, r, w0, b0, a.ymax, rt, mn, mx);
                } else {
                    if (!nw && nu == N / 64 && p.L[l + 1].nu == N / 32 && (N / 64) / G >= 4)
                        sp_cstr_c2<N>(in, r, w0, b0, a.ymax, rt.base, mn, mx);
                    else if (nw)
                        cf_body_cstr<RT_W>(in, r, nu, N / nu, w0, b0, a.ymax, rt, mn, mx, ilog2i(nu) - ilog2i(G));
                    else
                        cf_body_cstr<RT_C>(in, r, nu, N / nu, w0, b0, a.ymax, rt, mn, mx, ilog2i(nu) - ilog2i(G));
                }
                // the row's output range: every warp publishes its (min, max) (bits of outputs >= 0, -0 as
                // +0: bit order is value order, equal bits are equal values) to every rank
                {
                    const unsigned wmn = __reduce_min_sync(0xffffffffu, __float_as_uint(mn + 0.0f));
                    const unsigned wmx = __reduce_max_sync(0xffffffffu, __float_as_uint(mx + 0.0f));
                    if ((tid & 31) == 0) {
                        const int slot = (gl & 1) * G * kCWp + r * kCWp + (tid >> 5);
                        for (int h = 0; h < G; ++h) {
                            st_cl_u32(mapa_u32(smem_u32(s_vmn + slot), (uint32_t)h), wmn);
                            st_cl_u32(mapa_u32(smem_u32(s_vmx + slot), (uint32_t)h), wmx);
                        }
                    }
                }
                cluster_barrier();  // every rank's outputs, ranges (and the next row position) delivered
                unsigned rmn, rmx;
                {
                    const int ln = tid & 31;
                    unsigned m0 = 0xffffffffu, m1 = 0u;
                    for (int w = ln; w < G * kCWp; w += 32) {
                        m0 = min(m0, s_vmn[(gl & 1) * G * kCWp + w]);
                        m1 = max(m1, s_vmx[(gl & 1) * G * kCWp + w]);
                    }
                    rmn = __reduce_min_sync(0xffffffffu, m0);
                    rmx = __reduce_max_sync(0xffffffffu, m1);
                }
                ++full;
                ++gl;
                cur ^= 1;
                if (rmn == rmx) {  // constant row (R26) or dead (R23)
                    v = __uint_as_float(rmn);
                    if (a.const_skip) cst = true;
                    if (v == 0.0f && a.drop && dead_next) {
                        dead = true;
                        break;
                    }
                }
                // range prediction (R30, exact; kernels_pre_fused.cu): after k = t - l - 1 more layers every
                // element lies in [out^k(min), out^k(max)]; min >= thr_hi[k-1]: Y(t) is the constant row YMAX,
                // max <= thr_lo[k-1]: Y(t) is zero
                const int k2 = a.t - l - 1;
                if (a.thr_ok && k2 > 0) {
                    const int kk = min(k2, kRangeK);
                    if (__uint_as_float(rmn) >= p.thr_hi[kk - 1]) {
                        v = a.ymax;
                        cst = true;
                        break;
                    }
                    if (__uint_as_float(rmx) <= p.thr_lo[kk - 1]) {
                        v = 0.0f;
                        cst = true;
                        if (a.drop && a.dead_t) dead = true;
                        break;
                    }
                }
            } else {
                // constant row (R26): v' = sigma(chain(v) + b0), every rank evaluates the same scalar chain
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
                    break;
                }
            }
        }
        float* gslice = a.yout + (size_t)row * N + (size_t)r * kCS;
        if (dead && a.ydead) {
            float4* dz = reinterpret_cast<float4*>(a.ydead + (size_t)row * N + (size_t)r * kCS);
#pragma unroll
            for (int i = 0; i < kCS / 4 / T; ++i) dz[i * T + tid] = make_float4(0.f, 0.f, 0.f, 0.f);
        }
        if (!dead) {
            float4* d4 = reinterpret_cast<float4*>(gslice);
            if (cst) {
                const float4 v4 = make_float4(v, v, v, v);
#pragma unroll
                for (int i = 0; i < kCS / 4 / T; ++i) d4[i * T + tid] = v4;
            } else {  // the last layer's outputs: this rank's W slice in buffer `cur`
                const float4* s4 = reinterpret_cast<const float4*>(buf + cur * BS);
#pragma unroll
                for (int i = 0; i < kCS / 4 / T; ++i) d4[i * T + tid] = s4[i * T + tid];
            }
            if (r == 0 && tid == 0) {
                if (a.app_list) {
                    s_surv[nsurv++] = row;
                    if (nsurv == kCSurv) {
                        const int p0 = atomicAdd(a.app_count, nsurv);
                        for (int i = 0; i < nsurv; ++i) a.app_list[p0 + i] = s_surv[i];
                        nsurv = 0;
                    }
                }
                if (a.rconst && cst) {
                    a.rconst[row] = 1;
                    a.rval[row] = v;
                }
            }
        }
        if (r == 0 && tid == 0) {
            if (a.full_rl) atomicAdd(a.full_rl, (unsigned long long)full);
            if (a.n_const && cst) atomicAdd(a.n_const, 1);
        }
        // every rank is done with this row's buffers before any rank writes the next row's outputs (unless
        // the next row's first writes are halo-only, see end_barrier)
        if (end_barrier) cluster_barrier();
        pos = s_pos[(k + 1) & 1];
    }
    cluster_barrier();  // no CTA leaves while a peer may still access its shared memory
    if (r == 0 && tid == 0 && a.app_list && nsurv > 0) {
        const int p0 = atomicAdd(a.app_count, nsurv);
        for (int i = 0; i < nsurv; ++i) a.app_list[p0 + i] = s_surv[i];
    }
}

// ---------------------------------------------------------------------------- host side
// Class of layer l under the cluster kernel, or -1 when unsupported: N in {16384, 32768, 65536},
// uniform weight / bias circulant layers with 32 taps (checked by the caller via cls >= 0 of PF).
int pre_cluster_class(int N, int nu) {
    const int G = N / kCS;
    if (N % kCS != 0 || (G != 2 && G != 4 && G != 8) || nu < 1 || N % nu != 0) return -1;
    const int Q = N / nu;
    if ((nu & (nu - 1)) != 0) return -1;
    if (nu == 1) return CF_NU1;
    if (Q == 32) return (nu % G == 0) ? CF_Q32 : -1;
    if (nu >= 32 && Q / G >= 32 && Q % (2 * G) == 0 && (kCT % nu == 0) && 31 * nu <= 1024) return CF_WSTR;
    if (Q >= 64 && Q < 32 * G && (Q & (Q - 1)) == 0 && nu % G == 0 && (nu / G) * (Q / 32) == kCT) return CF_CSTR;
    return -1;
}
bool pre_cluster_supported(int N) {
    const int G = N / kCS;
    return N % kCS == 0 && (G == 2 || G == 4 || G == 8);
}
size_t pre_cluster_smem(int N, int Hh) {
    const int G = N / kCS;
    return sizeof(float) * 2 * (size_t)(kCS + Hh) + 2 * sizeof(uint64_t) + 2 * sizeof(int) +
           2 * (size_t)G * kCWp * (sizeof(int) + sizeof(float)) + 2 * (size_t)G * sizeof(uint32_t) +
           sizeof(uint32_t) * (size_t)((kCS + 1024) / 32) + sizeof(int) * kCSurv +
           2 * (size_t)G * kCWp * sizeof(unsigned);
}

template <int N, bool WUNI>
static cudaError_t launch_cl(const CfParams& p, int num_sms, cudaStream_t st) {
    constexpr int G = N / kCS;
    const size_t smem = pre_cluster_smem(N, p.Hh);
    auto kern = pre_cluster_kernel<N, WUNI>;
    int bps = 0;
    cudaError_t e = blocks_per_sm((const void*)kern, kCT, smem, &bps);
    if (e != cudaSuccess) return e;
    if (bps < 1) return cudaErrorInvalidConfiguration;
    cudaLaunchConfig_t cfg = {};
    int nclusters = 0;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = G;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.blockDim = dim3(kCT, 1, 1);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cfg.gridDim = dim3(G, 1, 1);
    e = cudaOccupancyMaxActiveClusters(&nclusters, (const void*)kern, &cfg);
    if (e != cudaSuccess) return e;
    if (nclusters < 1) return cudaErrorInvalidConfiguration;
    cfg.gridDim = dim3(G * nclusters, 1, 1);  // persistent clusters, rows scheduled dynamically
    e = cudaLaunchKernelEx(&cfg, kern, p);
    if (e != cudaSuccess) return e;
    return cudaGetLastError();
}

cudaError_t launch_pre_cluster(const PreFusedArgs& a, const PreFusedLayer* layers, int num_sms, cudaStream_t st) {
    if (a.t < 1 || a.t > kCfMaxLayers || !pre_cluster_supported(a.N)) return cudaErrorInvalidValue;
    static thread_local CfParams p;  // 32 KB: not on the stack
    p.a = a;
    int Hh = 64;
    for (int l = 0; l < a.t; ++l) {
        const int cls = pre_cluster_class(a.N, layers[l].nu);
        if (cls < 0) return cudaErrorInvalidValue;
        p.L[l].w0 = layers[l].w0;
        p.L[l].b0 = layers[l].b0;
        p.L[l].nu = layers[l].nu;
        p.L[l].flags = (cls & 15) | (layers[l].dead_next ? 16 : 0) | (layers[l].ymax_fixed ? 32 : 0);
        if (cls == CF_WSTR) Hh = Hh > 31 * layers[l].nu ? Hh : 31 * layers[l].nu;
    }
    p.L[a.t] = CfLayer{0.f, 0.f, 1, CF_NU1};
    // range prediction horizon tables (R30, kernels_const.cu), as launch_pre_fused
    p.a.thr_ok = a.const_skip && a.range_pred && range_tables(layers, a.t, a.ymax, p.thr_hi, p.thr_lo);
    p.a.dead_t = layers[a.t - 1].dead_next;
    p.Hh = (Hh + 127) / 128 * 128;  // bulk copies of the halo (fp32 and packed bits) in 16-byte multiples
    if (p.Hh > 1024) return cudaErrorInvalidValue;
    if (a.ybits && !((p.L[0].flags & 15) == CF_NU1 || (p.L[0].flags & 15) == CF_WSTR)) return cudaErrorInvalidValue;
    bool wuni = true;
    for (int l = 1; l < a.t; ++l) wuni = wuni && memcmp(&p.L[l].w0, &p.L[0].w0, sizeof(float)) == 0;
    switch (a.N) {
        case 16384: return wuni ? launch_cl<16384, true>(p, num_sms, st) : launch_cl<16384, false>(p, num_sms, st);
        case 32768: return wuni ? launch_cl<32768, true>(p, num_sms, st) : launch_cl<32768, false>(p, num_sms, st);
        case 65536: return wuni ? launch_cl<65536, true>(p, num_sms, st) : launch_cl<65536, false>(p, num_sms, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace snicit
