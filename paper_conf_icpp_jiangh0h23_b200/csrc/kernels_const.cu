// kernels_const.cu -- constant rows in the per-layer pre-convergence path (reading R26), sm_100a.
//
// A circulant layer with uniform weight and bias maps a row whose elements are all equal to v to the
// constant row sigma(chain(v) + b0) (every output evaluates the same stored-order fma chain on the
// same values, R12).  In constant-row mode the column-streaming and segmented layer kernels report
// each row's output range (min, max); a row with min == max leaves the active list for a constant
// list (row, value, layer), so later layers neither read nor write it.  At t, const_finish carries
// each constant row through the remaining layers with one scalar chain per layer and writes it once.
// Exact: results are bit-identical to the full evaluation (tested).
#include <cuda_runtime.h>

#include <cmath>
#include <cstring>

#include "snicit_internal.cuh"

namespace snicit {

// After a segmented layer: per list position, the row's (min, max) output bits (restored to the
// initial 0xffffffff / 0) decide constant -> constant list (or dead), else -> next active list
// (unordered, R24; warp-aggregated appends).
__global__ void const_split_kernel(const int* list_in, const int* count_in, unsigned* cmin, unsigned* cmax,
                                   int* list_out, int* count_out, int* clist, float* cval, int* clayer, int* ccount,
                                   int layer, int dead_drop, float thr_hi, float thr_lo, int thr_layer, int thr_dead,
                                   float ymax) {
    const int n = *count_in;
    const int lane = threadIdx.x & 31;
    for (int i0 = blockIdx.x * blockDim.x; i0 < n; i0 += gridDim.x * blockDim.x) {
        const int i = i0 + threadIdx.x;
        bool keep = false, cst = false;
        int row = 0, cl = layer;
        float v = 0.0f;
        if (i < n) {
            row = list_in[i];
            const unsigned umn = cmin[i], umx = cmax[i];
            cmin[i] = 0xffffffffu;
            cmax[i] = 0u;
            if (umn == umx) {
                v = __uint_as_float(umn);
                cst = !(v == 0.0f && dead_drop);
            } else if (__uint_as_float(umn) >= thr_hi) {  // R30: YMAX at t
                v = ymax;
                cst = true;
                cl = thr_layer;
            } else if (__uint_as_float(umx) <= thr_lo) {  // R30: zero at t
                cst = !thr_dead;
                cl = thr_layer;
            } else {
                keep = true;
            }
        }
        const unsigned mk = __ballot_sync(0xffffffffu, keep);
        int base = 0;
        if (lane == 0 && mk) base = atomicAdd(count_out, __popc(mk));
        base = __shfl_sync(0xffffffffu, base, 0);
        if (keep) list_out[base + __popc(mk & ((1u << lane) - 1u))] = row;
        if (cst) {
            const int p = atomicAdd(ccount, 1);
            clist[p] = row;
            cval[p] = v;
            clayer[p] = cl;
        }
    }
}

cudaError_t launch_const_split(const int* list_in, const int* count_in, unsigned* cmin, unsigned* cmax, int* list_out,
                               int* count_out, int* clist, float* cval, int* clayer, int* ccount, int layer,
                               int dead_drop, int max_rows, cudaStream_t st, const LayerArgs* thr) {
    int grid = max_rows > 0 ? (max_rows + 255) / 256 : 1;
    if (grid > 2048) grid = 2048;
    const_split_kernel<<<grid, 256, 0, st>>>(list_in, count_in, cmin, cmax, list_out, count_out, clist, cval, clayer,
                                             ccount, layer, dead_drop, thr ? thr->thr_hi : INFINITY,
                                             thr ? thr->thr_lo : -1.0f, thr ? thr->thr_layer : layer,
                                             thr ? thr->thr_dead : 0, thr ? thr->ymax : 0.0f);
    return cudaGetLastError();
}

bool range_tables(const PreFusedLayer* layers, int t, float ymax, float* hi, float* lo) {
    if (t < 1 || !(layers[0].w0 >= 0.0f)) return false;
    for (int l = 1; l < t; ++l)
        if (memcmp(&layers[l].w0, &layers[0].w0, sizeof(float)) != 0 ||
            memcmp(&layers[l].b0, &layers[0].b0, sizeof(float)) != 0)
            return false;
    const float w0 = layers[0].w0, b0 = layers[0].b0;
    auto out = [&](float m) {  // the kernels' chain for a constant input m (acc = fma(m, w0, acc) x 32), + b0, sigma
        float acc = 0.0f;
        for (int n = 0; n < 32; ++n) acc = std::fma(m, w0, acc);
        const float z = acc + b0;
        return std::fmin(std::fmax(z, 0.0f), ymax);
    };
    auto bits = [](float f) { uint32_t u; memcpy(&u, &f, 4); return u; };
    auto flt = [](uint32_t u) { float f; memcpy(&f, &u, 4); return f; };
    // out is non-decreasing on [0, ymax], so {m : out^k(m) == ymax} = [hi[k-1], ymax] with hi[k-1] = least m
    // with out(m) >= hi[k-2] (hi[-1] = ymax), and {m : out^k(m) == 0} = [0, lo[k-1]] with lo[k-1] = greatest
    // m with out(m) <= lo[k-2] (lo[-1] = 0); bisection over the bit patterns of [0, ymax] (order-preserving
    // for floats >= 0)
    const bool hi_ok = out(ymax) == ymax, lo_ok = out(0.0f) == 0.0f;
    float hprev = ymax, lprev = 0.0f;
    for (int k = 0; k < kRangeK; ++k) {
        hi[k] = INFINITY;
        lo[k] = -1.0f;
        if (hi_ok) {
            uint32_t a0 = 0, a1 = bits(ymax);
            while (a0 < a1) {
                const uint32_t mid = a0 + (a1 - a0) / 2;
                if (out(flt(mid)) >= hprev) a1 = mid; else a0 = mid + 1;
            }
            hi[k] = hprev = flt(a0);
        }
        if (lo_ok) {
            uint32_t a0 = 0, a1 = bits(ymax);
            while (a0 < a1) {
                const uint32_t mid = a0 + (a1 - a0 + 1) / 2;
                if (out(flt(mid)) <= lprev) a0 = mid; else a1 = mid - 1;
            }
            lo[k] = lprev = flt(a0);
        }
    }
    return hi_ok || lo_ok;
}

// At t: each constant row (value v after layer clayer) through layers clayer + 1 .. t - 1 by one scalar
// chain per layer (chain(+-0) = +0; chain(YMAX) precomputed on the host, ymax_fixed); dead rows (R23)
// vanish, the others are written (N values) and appended to the live list.
__global__ void __launch_bounds__(256) const_finish_kernel(const int* clist, const float* cval, const int* clayer,
                                                           const int* ccount, const PreFusedLayer* layers, int t,
                                                           float ymax, int drop, int N, float* y, int* live,
                                                           int* live_count, uint8_t* rconst, float* rval) {
    __shared__ float s_v;
    __shared__ int s_alive;
    const int n = *ccount;
    for (int e = blockIdx.x; e < n; e += gridDim.x) {
        if (threadIdx.x == 0) {
            float v = cval[e];
            bool alive = true;
            for (int l = clayer[e] + 1; l < t; ++l) {
                const PreFusedLayer d = layers[l];
                if (v == 0.0f) {
                    v = sigma(0.0f + d.b0, ymax);
                } else if (!(v == ymax && d.ymax_fixed)) {
                    float acc = 0.0f;
#pragma unroll
                    for (int k = 0; k < 32; ++k) acc = fmaf(v, d.w0, acc);
                    v = sigma(acc + d.b0, ymax);
                }
                if (v == 0.0f && drop && d.dead_next) {
                    alive = false;
                    break;
                }
            }
            s_v = v;
            s_alive = alive;
            if (alive) {
                live[atomicAdd(live_count, 1)] = clist[e];
                if (rconst) {
                    rconst[clist[e]] = 1;
                    rval[clist[e]] = v;
                }
            }
        }
        __syncthreads();
        if (s_alive) {
            float4* dst = reinterpret_cast<float4*>(y + (size_t)clist[e] * N);
            const float v = s_v;
            const float4 v4 = make_float4(v, v, v, v);
            for (int j = threadIdx.x; j < N / 4; j += blockDim.x) dst[j] = v4;
            for (int j = (N / 4) * 4 + threadIdx.x; j < N; j += blockDim.x) y[(size_t)clist[e] * N + j] = v;
        }
        __syncthreads();
    }
}

cudaError_t launch_const_finish(const int* clist, const float* cval, const int* clayer, const int* ccount,
                                const PreFusedLayer* layers, int t, float ymax, int drop, int N, float* y, int* live,
                                int* live_count, int num_sms, cudaStream_t st, uint8_t* rconst, float* rval) {
    const_finish_kernel<<<num_sms * 8, 256, 0, st>>>(clist, cval, clayer, ccount, layers, t, ymax, drop, N, y, live,
                                                     live_count, rconst, rval);
    return cudaGetLastError();
}

}  // namespace snicit
