// kernels_pre_pair.cu -- row-resident pre-convergence phase (a1) in the paired-half layout, sm_100a.
//
// The computation of kernels_pre_fused.cu (Eq. 1: layers 0..t-1 of a row kept in shared
// memory, the stored-order fma chains of R12 evaluated two at a time with packed FFMA2, constant rows
// R26, dead rows R23), with the row stored as PAIRS z[p] = (y[p], y[p + N/2]), p < N/2.  Every stride
// class of the SDGC layers pairs output q with output q + N/2:
//   NU1  (nu == 1):  thread i owns pairs p = 16 i + m, m < 16; its window is pairs 16 i .. 16 i + 46;
//   STR  (nu >= 32, Q = N/nu >= 64): item (c, a0) owns pairs (a0 + m) nu + c; window (a0 + j) nu + c;
//   Q32  (nu == N/32): thread c owns the residue class c -- pairs k nu + c, k < 16 (and, swapped, 16..31);
// so one 8-byte shared load fetches both FFMA2 operands of a window element (half the load instructions
// of the split layout, and no register packing), and one 8-byte store writes an output pair.  Pair p sits
// in slot p + (p >> 4) (one pad slot per 16): a half-warp's 16 lanes then touch 16 distinct 8-byte bank
// pairs in every class (lane strides 17, 1 and 1 slots), and every window offset is a compile-time
// immediate (the thread's base slot + j * 17 nu / 16).  Windows never wrap: pairs N/2 .. N/2 + Hp - 1 hold
// the swapped head pairs (y[p + N/2], y[p]) -- pair p + N/2 of the same definition, indices mod N -- copied
// after each layer by the threads that own pairs p < Hp.
// Results are bit-identical to the split layout and the oracle (the same chains; tested).
#include <cuda_runtime.h>

#include <cstring>

#include "snicit_internal.cuh"

namespace snicit {

typedef unsigned long long u64;
constexpr int kPpSurv = 32;

__device__ __forceinline__ int zsw(int p) { return p + (p >> 4); }  // slot of pair p
__device__ __forceinline__ u64 swap2(u64 v) { return (v >> 32) | (v << 32); }
__host__ __device__ inline int pp_slots(int pairs) { return pairs + (pairs + 15) / 16; }

// output pair at slot s: store, range update
__device__ __forceinline__ void pp_emit(u64* __restrict__ zs, float o1, float o2, float& mn, float& mx) {
    *zs = f2_pack(o1, o2);
    mn = fminf(mn, fminf(o1, o2));
    mx = fmaxf(mx, fmaxf(o1, o2));
}
// the swapped copies of this thread's output pairs p0 + m * step (m < 16) that lie in the head (p < Hp)
__device__ __forceinline__ void pp_halo(u64* __restrict__ zout, int p0, int step, int n2, int Hp) {
    if (p0 < Hp) {
#pragma unroll
        for (int m = 0; m < 16; ++m) {
            const int p = p0 + m * step;
            if (p < Hp) zout[zsw(n2 + p)] = swap2(zout[zsw(p)]);
        }
    }
}

template <int T>
__device__ __forceinline__ void pp_body_nu1(const u64* __restrict__ zin, u64* __restrict__ zout, float w0, float b0,
                                            float ymax, int Hp, float& mn, float& mx) {
    constexpr int N2 = 16 * T;
    const int p0 = 16 * (int)threadIdx.x;
    const u64* zi = zin + 17 * (int)threadIdx.x;  // slot of pair p0 + j = 17 i + j + (j >> 4)
    u64 W[47];
#pragma unroll
    for (int j = 0; j < 47; ++j) W[j] = zi[j + (j >> 4)];
    const u64 W2 = f2_pack(w0, w0), B2 = f2_pack(b0, b0);
    u64* zo = zout + 17 * (int)threadIdx.x;
#pragma unroll
    for (int m = 0; m < 16; ++m) {
        u64 acc = 0ull;
#pragma unroll
        for (int n = 0; n < 32; ++n) acc = f2_fma(W[m + n], W2, acc);
        float z1, z2;
        f2_unpack(f2_add(acc, B2), z1, z2);
        pp_emit(zo + m, sigma(z1, ymax), sigma(z2, ymax), mn, mx);
    }
    pp_halo(zout, p0, 1, N2, Hp);
}

// NU > 0: compile-time stride; 0: runtime
template <int T, int NU>
__device__ __forceinline__ void pp_body_str(const u64* __restrict__ zin, u64* __restrict__ zout, int nu_rt, float w0,
                                            float b0, float ymax, int Hp, float& mn, float& mx) {
    constexpr int N2 = 16 * T;
    const int nu = NU ? NU : nu_rt;
    const int c = (int)threadIdx.x % nu;
    const int a0 = ((int)threadIdx.x / nu) * 16;
    const int base = a0 * nu + c;
    // nu is a multiple of 16: slot(base + j nu) = zsw(base) + j * 17 nu / 16
    const int sb = zsw(base), sn = 17 * (nu >> 4);
    u64 W[47];
#pragma unroll
    for (int j = 0; j < 47; ++j) W[j] = zin[sb + j * sn];
    const u64 W2 = f2_pack(w0, w0), B2 = f2_pack(b0, b0);
#pragma unroll
    for (int m = 0; m < 16; ++m) {
        u64 acc = 0ull;
#pragma unroll
        for (int n = 0; n < 32; ++n) acc = f2_fma(W[m + n], W2, acc);
        float z1, z2;
        f2_unpack(f2_add(acc, B2), z1, z2);
        pp_emit(zout + sb + m * sn, sigma(z1, ymax), sigma(z2, ymax), mn, mx);
    }
    pp_halo(zout, base, nu, N2, Hp);
}

template <int T>
__device__ __forceinline__ void pp_body_q32(const u64* __restrict__ zin, u64* __restrict__ zout, float w0, float b0,
                                            float ymax, int Hp, float& mn, float& mx) {
    constexpr int N2 = 16 * T;
    constexpr int nu = T;  // Q == 32
    const int c = threadIdx.x;
    u64 P[16], S[16];  // P[k] = (y[k nu + c], y[(k + 16) nu + c]); S[k] = swapped = the pair of index k + 16
    const int sb = zsw(c), sn = 17 * (nu >> 4);  // slot(k nu + c) = zsw(c) + k * 17 nu / 16 (nu % 16 == 0)
#pragma unroll
    for (int k = 0; k < 16; ++k) P[k] = zin[sb + k * sn];
#pragma unroll
    for (int k = 0; k < 16; ++k) S[k] = swap2(P[k]);
    const u64 W2 = f2_pack(w0, w0), B2 = f2_pack(b0, b0);
#pragma unroll
    for (int m = 0; m < 16; ++m) {
        u64 acc = 0ull;
#pragma unroll
        for (int n = 0; n < 32; ++n) {
            const int k = (m + n) & 31;
            acc = f2_fma(k < 16 ? P[k] : S[k - 16], W2, acc);
        }
        float z1, z2;
        f2_unpack(f2_add(acc, B2), z1, z2);
        pp_emit(zout + sb + m * sn, sigma(z1, ymax), sigma(z2, ymax), mn, mx);
    }
    pp_halo(zout, c, nu, N2, Hp);
}

// linear row (float x[N]) or packed bits -> pairs z[0 .. N/2 + Hp) (indices mod N)
template <int T>
__device__ __forceinline__ void pp_fill(u64* __restrict__ z, const float* __restrict__ x, const uint32_t* bits,
                                        float one, int Hp) {
    constexpr int N = 32 * T, N2 = N / 2;
    for (int p = threadIdx.x; p < N2 + Hp; p += T) {
        const int k1 = p < N ? p : p - N;
        const int k2 = p + N2 < N ? p + N2 : p + N2 - N;
        float v1, v2;
        if (bits) {
            v1 = ((bits[k1 >> 5] >> (k1 & 31)) & 1u) ? one : 0.0f;
            v2 = ((bits[k2 >> 5] >> (k2 & 31)) & 1u) ? one : 0.0f;
        } else {
            v1 = x[k1];
            v2 = x[k2];
        }
        z[zsw(p)] = f2_pack(v1, v2);
    }
}

template <int T>
constexpr int kPpBufs = T >= 512 ? 3 : 2;  // a third buffer (linear staging) receives the next row
template <int T>
struct PpCfg {
    static constexpr int kMinBlocks = T <= 32 ? 16 : (T <= 64 ? 8 : (T <= 128 ? 4 : (T <= 256 ? 2 : 1)));
};

struct PpLayerParam {
    float w0, b0;
    int nu;
    int flags;  // cls | dead_next << 4 | ymax_fixed << 5
};
struct PrePairParams {
    PreFusedArgs a;  // a.H: halo in PAIRS (Hp)
    PpLayerParam L[kPfMaxLayers];
};
static_assert(sizeof(PrePairParams) <= 32764, "kernel parameter space");

size_t pre_pair_smem(int N, int Hp) {
    const int T = N / 32;
    const size_t zbytes = 8 * (size_t)pp_slots(N / 2 + Hp);
    const size_t stage = T >= 512 ? 4 * (size_t)N : 0;
    return 2 * zbytes + stage + 2 * sizeof(uint64_t) + 4 * sizeof(int) + 4 * sizeof(int) * (N / 32 / 32) +
           2 * sizeof(uint32_t) * (size_t)(N / 32) + sizeof(int) * kPpSurv;
}

template <int T, bool GENSTR, bool WUNI>
__global__ void __launch_bounds__(T, PpCfg<T>::kMinBlocks) pre_pair_kernel(const __grid_constant__ PrePairParams p) {
    const PreFusedArgs& a = p.a;
    constexpr int N = 32 * T, N2 = N / 2;
    constexpr int NB = kPpBufs<T>;
    extern __shared__ __align__(128) unsigned char smem[];
    const int Hp = a.H;
    const int ZS = pp_slots(N2 + Hp);  // slots per z buffer
    u64* const zb = reinterpret_cast<u64*>(smem);                          // [2][ZS]
    float* const stage = reinterpret_cast<float*>(zb + 2 * ZS);            // NB == 3: [N] next row (linear)
    uint64_t* bar = reinterpret_cast<uint64_t*>(stage + (NB == 3 ? N : 0));  // [2] row loads
    int* s_pos = reinterpret_cast<int*>(bar + 2);
    constexpr int kWarps = T / 32;
    float* s_rep = reinterpret_cast<float*>(s_pos + 4);
    int* s_ok = reinterpret_cast<int*>(s_rep + 2 * kWarps);
    uint32_t* s_bits = reinterpret_cast<uint32_t*>(s_ok + 2 * kWarps);  // [2][N/32]
    int* s_surv = reinterpret_cast<int*>(s_bits + 2 * (N / 32));
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
    int nsurv = 0;
    auto flush_surv = [&](bool force) {
        if (tid == 0 && nsurv > 0 && (force || nsurv == kPpSurv)) {
            const int p0 = atomicAdd(a.app_count, nsurv);
            for (int i = 0; i < nsurv; ++i) a.app_list[p0 + i] = s_surv[i];
            nsurv = 0;
        }
    };
    // row p_ -> linear destination `dst` (fp32) or the packed-bits slot, completion on bar[b]
    auto issue_load = [&](int p_, float* dst, int b) {
        const size_t r_ = (size_t)__ldg(a.rows + p_);
        if (a.ready) {  // streamed upload: wait until the copy engine has delivered this row's chunk
            const int* f = a.ready + (31 - __clz((int)(r_ / a.ready_rows) + 1));
            while (ld_acquire_gpu(f) == 0) __nanosleep(256);
            fence_proxy_async_global();
        }
        if (a.ybits) {
            mbar_arrive_expect_tx(&bar[b], (uint32_t)(N / 8));
            bulk_g2s(s_bits + b * (N / 32), a.ybits + r_ * (N / 32), N / 8, &bar[b]);
        } else {
            mbar_arrive_expect_tx(&bar[b], (uint32_t)(N * 4));
            bulk_g2s(dst, a.yin + r_ * N, N * 4, &bar[b]);
        }
    };
    uint32_t ph = 0;
    if (NB == 3 && tid == 0 && pos < count) issue_load(pos, stage, 0);
    int np = 0;
    for (int k = 0; pos < count; ++k) {
        const int row = __ldg(a.rows + pos);
        u64* zin = zb;
        u64* zout = zb + ZS;
        // NB == 2: the row lands (linear) in the second z buffer, which layer 0 overwrites
        float* lin = NB == 3 ? stage : reinterpret_cast<float*>(zout);
        if (tid == 0) {
            // generic-proxy accesses of the destination (previous row) ordered before the TMA write
            fence_proxy_async_smem();
            if (NB == 2) issue_load(pos, lin, k & 1);
            np = atomicAdd(a.work, 1);  // next row (consumed at the row end: latency hidden)
            if (NB == 3) s_pos[2 + (k & 1)] = np;
        }
        mbar_wait(&bar[k & 1], (ph >> (k & 1)) & 1u);
        ph ^= 1u << (k & 1);
        pp_fill<T>(zin, lin, a.ybits ? s_bits + (k & 1) * (N / 32) : nullptr, a.one, Hp);
        __syncthreads();  // pairs in place; the staging buffer is free
        if (NB == 3 && tid == 0 && np < count) {  // behind this row's compute
            fence_proxy_async_smem();
            issue_load(np, stage, (k + 1) & 1);
        }
        bool cst = false, dead = false;
        float v = 0.0f;
        int full = 0;
        int lend = a.t;  // the layer that zeroed the row (dead), or t
        for (int l = 0; l < a.t; ++l) {
            const float w0 = WUNI ? p.L[0].w0 : p.L[l].w0, b0 = p.L[l].b0;
            const int fl = p.L[l].flags;
            const bool dead_next = (fl >> 4) & 1;
            if (!cst) {
                float mn = __int_as_float(0x7f800000), mx = -__int_as_float(0x7f800000);
                const int cls = fl & 15;
                if (cls == PF_NU1)
                    pp_body_nu1<T>(zin, zout, w0, b0, a.ymax, Hp, mn, mx);
                else if (cls == PF_Q32)
                    pp_body_q32<T>(zin, zout, w0, b0, a.ymax, Hp, mn, mx);
                else if (GENSTR && p.L[l].nu != 32)
                    pp_body_str<T, 0>(zin, zout, p.L[l].nu, w0, b0, a.ymax, Hp, mn, mx);
                else
                    pp_body_str<T, 32>(zin, zout, 32, w0, b0, a.ymax, Hp, mn, mx);
                {  // "all outputs equal" in one barrier (warp votes published before it, kernels_pre_fused.cu)
                    const float ref = __shfl_sync(0xffffffffu, mn, 0);
                    const bool ok = __all_sync(0xffffffffu, mn >= ref && mx <= ref);
                    if ((tid & 31) == 0) {
                        s_rep[(l & 1) * kWarps + (tid >> 5)] = ref;
                        s_ok[(l & 1) * kWarps + (tid >> 5)] = ok ? 1 : 0;
                    }
                }
                __syncthreads();
                bool all_eq = true;
                const float o0 = s_rep[(l & 1) * kWarps];
#pragma unroll
                for (int w = 0; w < kWarps; ++w)
                    all_eq = all_eq && s_ok[(l & 1) * kWarps + w] && s_rep[(l & 1) * kWarps + w] == o0;
                ++full;
                u64* tz = zin;
                zin = zout;
                zout = tz;
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
                // constant row (R26): v' = sigma(chain(v) + b0); chain(+-0) = +0, chain(YMAX) on the host
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
            }
        }
        if (dead && a.ydead) {
            float4* dz = reinterpret_cast<float4*>(a.ydead + (size_t)row * N);
#pragma unroll
            for (int i = 0; i < N / 4 / T; ++i) dz[i * T + tid] = make_float4(0.f, 0.f, 0.f, 0.f);
        }
        if (!dead) {
            float* gout = a.yout + (size_t)row * N;
            if (cst) {
                const float4 v4 = make_float4(v, v, v, v);
#pragma unroll
                for (int i = 0; i < N / 4 / T; ++i) reinterpret_cast<float4*>(gout)[i * T + tid] = v4;
            } else {  // the last layer's pairs -> the two halves of the row (coalesced per warp)
#pragma unroll 4
                for (int q = tid; q < N2; q += T) {
                    float lo, hi;
                    f2_unpack(zin[zsw(q)], lo, hi);
                    gout[q] = lo;
                    gout[q + N2] = hi;
                }
            }
            if (tid == 0 && a.app_list) {
                s_surv[nsurv++] = row;
                flush_surv(false);
            }
            if (tid == 0 && a.rconst && cst) {
                a.rconst[row] = 1;
                a.rval[row] = v;
            }
        }
        if (tid == 0) {
            if (a.full_rl) atomicAdd(a.full_rl, (unsigned long long)full);
            if (a.n_const && cst) atomicAdd(a.n_const, 1);
            if (a.dyn) {
                atomicAdd(a.dyn + full, 1ull);
                atomicAdd(a.dyn + (a.t + 1) + lend, 1ull);
            }
        }
        if (NB == 2 && tid == 0) {
            s_pos[2 + (k & 1)] = np;
            if (np < count && a.l2_prefetch && !a.ybits)
                bulk_prefetch_l2(a.yin + (size_t)__ldg(a.rows + np) * N, N * 4);
        }
        __syncthreads();  // buffers free, next position visible
        pos = s_pos[2 + (k & 1)];
    }
    if (a.app_list) flush_surv(true);
}

template <int T, bool GENSTR, bool WUNI>
static cudaError_t launch_pp_tg(const PrePairParams& p, int num_sms, cudaStream_t st) {
    const size_t smem = pre_pair_smem(p.a.N, p.a.H);
    int bps = 0;
    cudaError_t e = blocks_per_sm((const void*)pre_pair_kernel<T, GENSTR, WUNI>, T, smem, &bps);
    if (e != cudaSuccess) return e;
    if (bps < 1) return cudaErrorInvalidConfiguration;
    pre_pair_kernel<T, GENSTR, WUNI><<<num_sms * bps, T, smem, st>>>(p);
    return cudaGetLastError();
}
template <int T>
static cudaError_t launch_pp_t(const PrePairParams& p, bool wuni, int num_sms, cudaStream_t st) {
    if (p.a.gen_str) return wuni ? launch_pp_tg<T, true, true>(p, num_sms, st) : launch_pp_tg<T, true, false>(p, num_sms, st);
    return wuni ? launch_pp_tg<T, false, true>(p, num_sms, st) : launch_pp_tg<T, false, false>(p, num_sms, st);
}

// halo pairs for layers 0..t-1: 31 past a window (nu == 1) or 31 nu (strided), multiple of 16
int pre_pair_halo(int N, const PreFusedLayer* layers, int t) {
    int hp = 32;
    for (int l = 0; l < t; ++l)
        if (layers[l].cls == PF_STR) hp = hp > 31 * layers[l].nu ? hp : 31 * layers[l].nu;
    hp = (hp + 15) / 16 * 16;
    return hp <= N / 2 ? hp : -1;  // halo pairs index y mod N: at most N/2 of them are distinct
}

cudaError_t launch_pre_pair(const PreFusedArgs& a, const PreFusedLayer* layers, int num_sms, cudaStream_t st) {
    if (a.t < 1 || a.t > kPfMaxLayers) return cudaErrorInvalidValue;
    static thread_local PrePairParams p;
    p.a = a;
    p.a.H = pre_pair_halo(a.N, layers, a.t);
    if (p.a.H < 0) return cudaErrorInvalidValue;
    p.a.l2_prefetch = 1;
    for (int l = 0; l < a.t; ++l) {
        p.L[l].w0 = layers[l].w0;
        p.L[l].b0 = layers[l].b0;
        p.L[l].nu = layers[l].nu;
        p.L[l].flags = (layers[l].cls & 15) | (layers[l].dead_next ? 16 : 0) | (layers[l].ymax_fixed ? 32 : 0);
    }
    bool wuni = true;
    for (int l = 1; l < a.t; ++l) wuni = wuni && memcmp(&p.L[l].w0, &p.L[0].w0, sizeof(float)) == 0;
    switch (pre_fused_threads(a.N)) {
        case 32: return launch_pp_t<32>(p, wuni, num_sms, st);
        case 64: return launch_pp_t<64>(p, wuni, num_sms, st);
        case 128: return launch_pp_t<128>(p, wuni, num_sms, st);
        case 256: return launch_pp_t<256>(p, wuni, num_sms, st);
        case 512: return launch_pp_t<512>(p, wuni, num_sms, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace snicit
