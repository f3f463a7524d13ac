// kernels_gen.cu -- general-CSC layer kernel with row-interleaved tiles and lanes over rows (sm_100a).
//
// Computes what layer_ell_kernel computes (Eq. 1, the stored-order fma chain of every output,
// R12; PLAIN / CENTROID / RESIDUAL epilogues of Eq. 5) for layers with no structure to exploit
// (random gathers).  Every fma of a gather kernel needs one input value delivered from shared
// memory to its lane, and the L1 / shared-memory data pipe delivers 128 B per clock per SM -- so the
// roofline is 32 fmas/clk/SM (a quarter of the FP32 pipe), and EVERY byte a lane receives counts: a
// 16-byte per-lane index load costs as many pipe cycles as a 16-byte data load (ncu, round 2 (r02c): the first
// version of this kernel spent half of its data-pipe wavefronts on index loads).  Hence:
//  * a tile holds RL rows interleaved (element (k, r) at k RL + r) and every lane owns FOUR consecutive
//    rows: one 16-byte shared load (LDS.128) feeds two packed FFMA2 of the same tap, so an index (u16,
//    eight taps per 16-byte load) is paid once per four fmas;
//  * a warp instruction covers G outputs x (32 / G) lanes x 4 rows (RL = 128 / G): G = 2 (N <= 384) and
//    G = 4 (N <= 1536) read whole 128-byte lines per quarter-warp -- conflict-free for ANY W; G = 16
//    (N <= 4864, 8-row tiles) reads four outputs' 32-byte segments per quarter-warp, conflict-free when
//    their inputs differ mod 4, which the load-time schedule arranges (gen_build_layer: quads of outputs
//    with disjoint bank groups tap by tap; exact for shift-structured W, greedy otherwise);
//  * G = 16 stages outputs per warp (scheduled outputs are not contiguous) and writes row segments;
//    G = 2 / 4 lanes own U consecutive outputs and store them as float4 per row;
//  * padded taps (K not a multiple of 8, ragged columns) read a zero input slot (k = N) with weight 0:
//    exact, since fma(0, 0, acc) = acc for every acc != -0 and a chain started at +0 is never -0 (RN).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <vector>

#include "snicit_internal.cuh"

namespace snicit {

namespace {
constexpr int kGenSurvCap = 256;
template <int G>
constexpr int kGenRL = 128 / G;  // rows per tile (G = 2, 4, 16)
template <int G>
constexpr int kGenThreads = G == 16 ? 512 : 256;
template <int G>
constexpr int kGenU = G == 16 ? 2 : 4;  // output groups per lane in flight
template <int G>
constexpr int kGenMinBlocks = G == 16 ? 1 : 2;  // G = 2 / 4: two CTAs per SM (<= 128 registers)
template <int G>
constexpr int kGenLogRB = G == 2 ? 8 : (G == 4 ? 7 : 5);  // log2(RL * 4): bytes per input k in the tile
constexpr int kGenStageStride = 132;  // G = 16 staging: 8 rows x 128 outputs (+4 pad) per warp

size_t gen_tile_bytes(int N, int G) { return (size_t)(N + 1) * (128 / G) * 4; }
size_t gen_smem_bytes(int N, int G) {
    const int nw = (G == 16 ? 512 : 256) / 32;
    const size_t stage = G == 16 ? (size_t)nw * 8 * kGenStageStride * 4 : 0;
    return gen_tile_bytes(N, G) + stage + 20 * (128 / G) + 4 * kGenSurvCap + 64;
}
}  // namespace

// Output group size G for a network of N neurons: 1, 4 or 16; 0 = kernel not used (previous ELL kernels).
int gen_rows_per_tile(int N) {
    if (N < 32 || N % 32 != 0 || N >= 65535) return 0;
    if (N <= 384 && gen_smem_bytes(N, 2) <= 110 * 1024) return 2;  // two CTAs per SM
    if (N <= 1536 && N % 128 == 0 && gen_smem_bytes(N, 4) <= 220 * 1024) return 4;
    if (N % 128 == 0 && gen_smem_bytes(N, 16) <= 220 * 1024) return 16;
    return 0;
}

// Load-time schedule of one layer.  cidx/cval: the stored inputs of every output column (chain order).
// A warp instruction serves one SET of G outputs (member q = lane group); set s, tap block b (8 taps),
// member q own the 8 u16 input ids at idx[((s * Kp8 + b) * G + q) * 8 ..] and the 8 weights at the same
// offset of w (when w != nullptr), so the G blocks a warp loads are contiguous (Kp8 = ceil(Kp / 8) blocks;
// Kp is a multiple of 4 and a last half block is skipped by the kernel).  Padded taps read the zero slot N
// with weight 0.  Sets: G = 2 / 4: unit t of 4 G outputs, set 4 t + u, member q = output 4 G t + 4 q + u
// (a lane's U = 4 outputs are consecutive: float4 stores); G = 16: the
// outputs of 128-output chunk c grouped into 32 quads with inputs in distinct bank groups (k & 3) tap by tap
// where possible (sched[c * 128 + 4 qd + m] = output id), set s = quads 4 s .. 4 s + 3.  Returns the mean
// shared-memory wavefronts per quarter-warp tap (1.0 = conflict-free; G = 2 / 4 read whole lines).
double gen_build_layer(int N, int G, int Kp, const std::vector<std::vector<int32_t>>& cidx,
                       const std::vector<std::vector<float>>& cval, uint16_t* idx, float* w, uint16_t* sched) {
    const int Kp8 = (Kp + 7) / 8;
    std::vector<int> order(N);  // output of slot p (set p / G, member p % G)
    if (G != 16) {  // U = 4 sets per unit of 4 G outputs; member q of set u takes output 4 q + u of the unit
        for (int set = 0; set < N / G; ++set)
            for (int q = 0; q < G; ++q) order[set * G + q] = (set / 4) * (4 * G) + q * 4 + set % 4;
    } else {
        // quads with disjoint bank groups tap by tap.  sig = 2-bit group of the first 32 taps (padded taps
        // read the broadcast zero slot: counted as group N & 3 = 0).
        const int T = std::min(Kp, 32);
        const uint64_t tmask = T >= 32 ? ~0ull : ((1ull << (2 * T)) - 1);
        const uint64_t lo = 0x5555555555555555ull & tmask;
        std::vector<uint64_t> sig(N);
        for (int j = 0; j < N; ++j) {
            uint64_t sg = 0;
            for (int n = 0; n < T && n < (int)cidx[j].size(); ++n) sg |= (uint64_t)(cidx[j][n] & 3) << (2 * n);
            sig[j] = sg;
        }
        auto eq = [&](int a, int b) {
            const uint64_t x = sig[a] ^ sig[b];
            return __builtin_popcountll(~(x | (x >> 1)) & lo);
        };
        std::vector<int> pool;
        for (int c = 0; c < N / 128; ++c) {
            pool.clear();
            for (int j = 0; j < 128; ++j) pool.push_back(c * 128 + j);
            for (int qd = 0; qd < 32; ++qd) {
                int pick[4];
                pick[0] = pool[0];
                pool.erase(pool.begin());
                for (int m = 1; m < 4; ++m) {
                    int best = 0, bc = 1 << 30;
                    for (int i = 0; i < (int)pool.size(); ++i) {
                        int cost = 0;
                        for (int p = 0; p < m; ++p) cost += eq(pick[p], pool[i]);
                        if (cost < bc) {
                            bc = cost;
                            best = i;
                            if (cost == 0) break;
                        }
                    }
                    pick[m] = pool[best];
                    pool.erase(pool.begin() + best);
                }
                for (int m = 0; m < 4; ++m) order[c * 128 + qd * 4 + m] = pick[m];
            }
        }
        for (int p = 0; p < N; ++p) sched[p] = (uint16_t)order[p];
    }
    // G <= 4: the tile's 16-byte units are XOR-swizzled (unit of input k, row quad rq at k RL/4 + (rq ^ s_k),
    // s_k = (k >> 2) & 7) so the transposed tile load is coalesced AND conflict-free; the entry holds
    // P_k = k RL/4 | s_k and a lane reads unit P_k ^ rq.  G = 16: the entry is k.
    auto ent = [&](int k) -> uint16_t {
        if (G == 16) return (uint16_t)k;
        return (uint16_t)((k * (32 / G)) | ((k >> 2) & 7));
    };
    for (int p = 0; p < N; ++p) {
        const int j = order[p], set = p / G, q = p % G;
        for (int n = 0; n < Kp8 * 8; ++n) {
            const size_t e = (((size_t)set * Kp8 + n / 8) * G + q) * 8 + n % 8;
            const bool real = n < (int)cidx[j].size();
            idx[e] = ent(real ? cidx[j][n] : N);
            if (w) w[e] = real ? cval[j][n] : 0.0f;
        }
    }
    if (G != 16) return 1.0;
    double tot = 0;
    size_t cnt = 0;
    for (int g = 0; g < N / 4; ++g)
        for (int n = 0; n < Kp; ++n) {
            int m[4] = {0, 0, 0, 0};
            int seen[4];
            int ns = 0;
            for (int q = 0; q < 4; ++q) {
                const int j = order[4 * g + q];
                const int k = n < (int)cidx[j].size() ? cidx[j][n] : N;
                bool dup = false;  // same address: broadcast
                for (int i = 0; i < ns; ++i) dup |= seen[i] == k;
                if (dup) continue;
                seen[ns++] = k;
                ++m[k & 3];
            }
            tot += *std::max_element(m, m + 4);
            ++cnt;
        }
    return cnt ? tot / cnt : 1.0;
}

// ------------------------------------------------------------------------------------------- kernel
template <int MODE, int G, bool UNIF>
__global__ void __launch_bounds__(kGenThreads<G>, kGenMinBlocks<G>) layer_gen_kernel(LayerArgs a) {
    constexpr int RL = kGenRL<G>, NT = kGenThreads<G>, NW = NT / 32, U = kGenU<G>, LOGRB = kGenLogRB<G>;
    constexpr int LPO = 32 / G;  // lanes per output (row quads)
    extern __shared__ __align__(128) unsigned char smem[];
    const int N = a.N, N4 = N >> 2, Kp8 = (a.gkp + 7) >> 3;
    const bool half_tail = (a.gkp & 7) != 0;  // the last 8-tap block holds 4 taps (+4 never evaluated)
    float* s_in = reinterpret_cast<float*>(smem);
    float* s_stage = reinterpret_cast<float*>(smem + (size_t)(N + 1) * RL * 4);
    int* s_flag = reinterpret_cast<int*>(s_stage + (G == 16 ? NW * 8 * kGenStageStride : 0));
    int* s_row = s_flag + RL;
    int* s_slot = s_row + RL;
    unsigned* s_cmn = reinterpret_cast<unsigned*>(s_slot + RL);
    unsigned* s_cmx = s_cmn + RL;
    int* s_surv = reinterpret_cast<int*>(s_cmx + RL);
    __shared__ int s_nsurv, s_pos;

    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (blockIdx.x == 0 && threadIdx.x == 0 && a.zero_count) *a.zero_count = 0;
    if (threadIdx.x == 0) s_nsurv = 0;
    if (threadIdx.x < RL) s_in[(size_t)N * RL + threadIdx.x] = 0.0f;  // the zero slot (k = N) of padded taps
    const int count = *a.count;
    const int ntiles = (count + RL - 1) / RL;
    // lane -> (output q within the warp instruction, row quad rq: rows 4 rq .. 4 rq + 3 of the tile)
    const int q = G == 16 ? (lane >> 1) : lane / LPO;
    const int rq = G == 16 ? (lane & 1) : lane % LPO;
    // G = 16: lane's rows at byte k*32 + rq*16; G <= 4: unit (P_k ^ rq) (swizzled, see gen_build_layer)
    const uint32_t sbase = smem_u32(s_in) + (G == 16 ? (uint32_t)rq * 16u : 0u);
    const uint4* gidx = reinterpret_cast<const uint4*>(a.gidx);
    const float4* gw = reinterpret_cast<const float4*>(a.gval);
    __syncthreads();
    for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const int r0 = tile * RL;
        const int nr = min(RL, count - r0);
        if (threadIdx.x < RL) {
            const int row = a.rows[r0 + min((int)threadIdx.x, nr - 1)];
            s_row[threadIdx.x] = row;
            s_flag[threadIdx.x] = 0;
            s_cmn[threadIdx.x] = 0xffffffffu;
            s_cmx[threadIdx.x] = 0u;
            if constexpr (MODE == MODE_RESIDUAL) s_slot[threadIdx.x] = a.cslot[row];
        } else if (threadIdx.x < 2 * RL) {  // the next tile's rows -> L2 while this one computes
            const int nt = tile + gridDim.x, i = threadIdx.x - RL;
            if (nt < ntiles && nt * RL + i < count)
                bulk_prefetch_l2(a.yin + (size_t)a.rows[nt * RL + i] * N, (uint32_t)N * 4);
        }
        __syncthreads();
        // transposed, conflict-free tile load
        if constexpr (G == 16) {
            // lanes: 8 rows x 4 consecutive chunks; step i stores component (i + cc) & 3 (bank groups distinct)
            for (int idx = threadIdx.x; idx < RL * N4; idx += NT) {
                const int rr = idx & 7, c = idx >> 3, cc = c & 3;
                const float4 v = __ldg(reinterpret_cast<const float4*>(a.yin + (size_t)s_row[rr] * N) + c);
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    const int comp = (i + cc) & 3;
                    const float x = comp == 0 ? v.x : comp == 1 ? v.y : comp == 2 ? v.z : v.w;
                    s_in[(4 * c + comp) * 8 + rr] = x;
                }
            }
        } else {
            // lanes: 4 rows x 8 consecutive float4 chunks (4 x 128-byte row segments); element (k, r) goes to
            // word 4 (k RL/4 + ((r >> 2) ^ s_k)) + (r & 3), s_k = (k >> 2) & 7 = c & 7: 32 distinct banks
            constexpr int NQ = RL / 4;
            for (int idx = threadIdx.x; idx < RL * N4; idx += NT) {
                const int cc = idx & 7, rho = (idx >> 3) & 3, blk = idx >> 5;
                const int rq4 = blk % NQ, c = 8 * (blk / NQ) + cc, rr = 4 * rq4 + rho;
                const float4 v = __ldg(reinterpret_cast<const float4*>(a.yin + (size_t)s_row[rr] * N) + c);
                float* d = s_in + (size_t)4 * ((size_t)(4 * c) * NQ + (rq4 ^ cc)) + rho;
                d[0] = v.x;
                d[4 * NQ] = v.y;
                d[8 * NQ] = v.z;
                d[12 * NQ] = v.w;
            }
        }
        __syncthreads();
        int my_row[4], my_slot[4];
        bool my_valid[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            my_row[i] = s_row[4 * rq + i];
            my_slot[i] = MODE == MODE_RESIDUAL ? s_slot[4 * rq + i] : 0;
            my_valid[i] = 4 * rq + i < nr;
        }
        unsigned anyr = 0;  // bit i: row 4 rq + i has a non-zero output in this lane's outputs
        unsigned rmn[4], rmx[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            rmn[i] = 0xffffffffu;
            rmx[i] = 0u;
        }
        // warp work unit: G * U outputs; a warp owns chunks of CHK outputs (G = 16: the 128 outputs its
        // staging tile collects, in 4 units of 32)
        constexpr int UNIT = G * U, CHK = G == 16 ? 128 : UNIT;
        for (int ck = warp * CHK; ck < N; ck += NW * CHK)
        for (int u0 = ck; u0 < ck + CHK; u0 += UNIT) {
            int jj[U];
#pragma unroll
            for (int u = 0; u < U; ++u)
                jj[u] = G == 16 ? (int)__ldg(a.gsched + u0 + u * 16 + q) : u0 + q * U + u;
            unsigned long long acc[U][2];
#pragma unroll
            for (int u = 0; u < U; ++u) acc[u][0] = acc[u][1] = 0ull;
            // set of instruction u: G = 1: output u0 + u; G = 4 / 16: (u0 / UNIT) * U + u
            const uint4* ip[U];
            const float4* wp[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const size_t set = (size_t)(u0 / UNIT) * U + u;
                ip[u] = gidx + set * Kp8 * G + q;
                wp[u] = gw + (set * Kp8 * G + q) * 2;
            }
            uint4 I[U];
#pragma unroll
            for (int u = 0; u < U; ++u) I[u] = __ldg(ip[u]);
#pragma unroll 1
            for (int b = 0; b < Kp8; ++b) {
                // next block's ids in flight while this block's 8 taps run (weights: this block's, loaded
                // here -- prefetching both needs more than the 128 registers of two CTAs per SM)
                const int bn = b + 1 < Kp8 ? b + 1 : b;
                uint4 In[U];
                float4 Wv[U][2];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    In[u] = __ldg(ip[u] + (size_t)bn * G);
                    if constexpr (!UNIF) {
                        Wv[u][0] = __ldg(wp[u] + (size_t)b * G * 2);
                        Wv[u][1] = __ldg(wp[u] + (size_t)b * G * 2 + 1);
                    }
                }
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    if (h == 1 && half_tail && b == Kp8 - 1) break;
#pragma unroll
                    for (int u = 0; u < U; ++u) {
                        const uint32_t p0 = h ? I[u].z : I[u].x, p1 = h ? I[u].w : I[u].y;
                        const uint32_t kk[4] = {p0 & 0xffffu, p0 >> 16, p1 & 0xffffu, p1 >> 16};
                        float ww[4];
                        if constexpr (UNIF) {
                            ww[0] = ww[1] = ww[2] = ww[3] = a.w0;
                        } else {
                            ww[0] = Wv[u][h].x;
                            ww[1] = Wv[u][h].y;
                            ww[2] = Wv[u][h].z;
                            ww[3] = Wv[u][h].w;
                        }
#pragma unroll
                        for (int i = 0; i < 4; ++i) {
                            float4 v;
                            asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                                         : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                                         : "r"(G == 16 ? sbase + (kk[i] << LOGRB)
                                                       : sbase + ((kk[i] ^ (uint32_t)rq) << 4)));
                            const unsigned long long W2 = f2_pack(ww[i], ww[i]);
                            acc[u][0] = f2_fma(f2_pack(v.x, v.y), W2, acc[u][0]);
                            acc[u][1] = f2_fma(f2_pack(v.z, v.w), W2, acc[u][1]);
                        }
                    }
                }
#pragma unroll
                for (int u = 0; u < U; ++u) I[u] = In[u];
            }
            // epilogue: v[u][i] for row 4 rq + i, output jj[u].  G = 2 / 4: a lane's U = 4 outputs are
            // consecutive, so bias, a_c (RESIDUAL) and a_out (CENTROID) move as one float4 per row
            float vo[U][4];
            float bv[U];
            float acv[4][U];  // RESIDUAL, G <= 4: a_c of row i, outputs jj[0..3]
            if constexpr (G != 16) {
                if (a.uniform_bias) {
#pragma unroll
                    for (int u = 0; u < U; ++u) bv[u] = __ldg(a.bias);
                } else {
                    const float4 b4 = __ldg(reinterpret_cast<const float4*>(a.bias + jj[0]));
                    bv[0] = b4.x;
                    bv[1] = b4.y;
                    bv[2] = b4.z;
                    bv[3] = b4.w;
                }
                if constexpr (MODE == MODE_RESIDUAL) {
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const float4 c4 = __ldg(reinterpret_cast<const float4*>(a.a_c + (size_t)my_slot[i] * N + jj[0]));
                        acv[i][0] = c4.x;
                        acv[i][1] = c4.y;
                        acv[i][2] = c4.z;
                        acv[i][3] = c4.w;
                    }
                }
            } else {
#pragma unroll
                for (int u = 0; u < U; ++u) bv[u] = a.uniform_bias ? __ldg(a.bias) : __ldg(a.bias + jj[u]);
            }
            float zc[4][U];  // CENTROID, G <= 4: pre-activations kept for one float4 store per row
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int j = jj[u];
                const float bj = bv[u];
                float z[4];
                f2_unpack(acc[u][0], z[0], z[1]);
                f2_unpack(acc[u][1], z[2], z[3]);
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    float v;
                    if constexpr (G != 16 && MODE == MODE_RESIDUAL) {  // Eq. 5 second case (as epilogue<>)
                        const float c = acv[i][u];
                        v = sigma((c + z[i]) + bj, a.ymax) - sigma(c + bj, a.ymax);
                        if (a.prune_eps > 0.0f && fabsf(v) <= a.prune_eps) v = 0.0f;
                    } else if constexpr (G != 16 && MODE == MODE_CENTROID) {  // Eq. 5 first case, a_c kept
                        zc[i][u] = z[i];
                        v = sigma(z[i] + bj, a.ymax);
                    } else {
                        v = epilogue<MODE>(a, z[i], bj, j, my_row[i], my_slot[i], my_valid[i]);
                    }
                    vo[u][i] = v;
                    if (my_valid[i]) {
                        if (v != 0.0f) anyr |= 1u << i;
                        if (MODE == MODE_PLAIN) {
                            const unsigned uv = __float_as_uint(v + 0.0f);
                            rmn[i] = min(rmn[i], uv);
                            rmx[i] = max(rmx[i], uv);
                        }
                    }
                }
            }
            if constexpr (G == 16) {
                // stage [8 rows][128 outputs of the chunk], then 8 coalesced 512-byte row segments
                float* stage = s_stage + warp * 8 * kGenStageStride;
                const int c0 = u0 & ~127;
#pragma unroll
                for (int u = 0; u < U; ++u)
#pragma unroll
                    for (int i = 0; i < 4; ++i) stage[(4 * rq + i) * kGenStageStride + (jj[u] - c0)] = vo[u][i];
                if (((u0 + UNIT) & 127) == 0) {  // the warp's chunk is complete
                    __syncwarp();
                    for (int rr = 0; rr < nr; ++rr)
                        reinterpret_cast<float4*>(a.yout + (size_t)s_row[rr] * N + c0)[lane] =
                            reinterpret_cast<const float4*>(stage + rr * kGenStageStride)[lane];
                    __syncwarp();
                }
            } else {
                // U = 4 consecutive outputs per lane: one float4 per row
#pragma unroll
                for (int i = 0; i < 4; ++i)
                    if (my_valid[i]) {
                        *reinterpret_cast<float4*>(a.yout + (size_t)my_row[i] * N + u0 + q * U) =
                            make_float4(vo[0][i], vo[1][i], vo[2][i], vo[3][i]);
                        if constexpr (MODE == MODE_CENTROID)
                            *reinterpret_cast<float4*>(a.a_out + (size_t)my_row[i] * N + u0 + q * U) =
                                make_float4(zc[i][0], zc[i][1], zc[i][2], zc[i][3]);
                    }
            }
        }
        // per-row aggregates: lanes of the same row quad combine, then one shared atomic per row
#pragma unroll
        for (int m = LPO; m < 32; m <<= 1) {
            anyr |= __shfl_xor_sync(0xffffffffu, anyr, m);
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                rmn[i] = min(rmn[i], __shfl_xor_sync(0xffffffffu, rmn[i], m));
                rmx[i] = max(rmx[i], __shfl_xor_sync(0xffffffffu, rmx[i], m));
            }
        }
        if (q == 0) {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                if (!my_valid[i]) continue;
                if (anyr & (1u << i)) s_flag[4 * rq + i] = 1;
                if (MODE == MODE_PLAIN && a.cmin) {
                    atomicMin(&s_cmn[4 * rq + i], rmn[i]);
                    atomicMax(&s_cmx[4 * rq + i], rmx[i]);
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
        if (a.app_list && s_nsurv > kGenSurvCap - RL) {
            if (threadIdx.x == 0) s_pos = atomicAdd(a.app_count, s_nsurv);
            __syncthreads();
            for (int i = threadIdx.x; i < s_nsurv; i += NT) a.app_list[s_pos + i] = s_surv[i];
            __syncthreads();
            if (threadIdx.x == 0) s_nsurv = 0;
            __syncthreads();
        }
    }
    if (a.app_list) {
        __syncthreads();
        const int n = s_nsurv;
        if (n > 0) {
            if (threadIdx.x == 0) s_pos = atomicAdd(a.app_count, n);
            __syncthreads();
            for (int i = threadIdx.x; i < n; i += NT) a.app_list[s_pos + i] = s_surv[i];
        }
    }
}

template <int MODE, int G>
static cudaError_t launch_gen_t(const LayerArgs& a, int max_rows, int num_sms, cudaStream_t st) {
    const size_t smem = gen_smem_bytes(a.N, G);
    void (*kern)(LayerArgs) = a.gval ? layer_gen_kernel<MODE, G, false> : layer_gen_kernel<MODE, G, true>;
    int per_sm = 1;
    cudaError_t e = blocks_per_sm((const void*)kern, kGenThreads<G>, smem, &per_sm);
    if (e != cudaSuccess) return e;
    const int tiles = (max_rows + kGenRL<G> - 1) / kGenRL<G>;
    int grid = num_sms * per_sm;
    if (grid > tiles) grid = tiles;
    if (grid < 1) grid = 1;
    kern<<<grid, kGenThreads<G>, smem, st>>>(a);
    return cudaGetLastError();
}

template <int G>
static cudaError_t launch_gen_g(const LayerArgs& a, int mode, int max_rows, int num_sms, cudaStream_t st) {
    switch (mode) {
        case MODE_PLAIN: return launch_gen_t<MODE_PLAIN, G>(a, max_rows, num_sms, st);
        case MODE_CENTROID: return launch_gen_t<MODE_CENTROID, G>(a, max_rows, num_sms, st);
        default: return launch_gen_t<MODE_RESIDUAL, G>(a, max_rows, num_sms, st);
    }
}

cudaError_t launch_layer_gen(const LayerArgs& a, int mode, int max_rows, int num_sms, cudaStream_t st) {
    if (max_rows <= 0) return cudaSuccess;
    switch (a.grl) {
        case 2: return launch_gen_g<2>(a, mode, max_rows, num_sms, st);
        case 4: return launch_gen_g<4>(a, mode, max_rows, num_sms, st);
        default: return launch_gen_g<16>(a, mode, max_rows, num_sms, st);
    }
}

}  // namespace snicit
