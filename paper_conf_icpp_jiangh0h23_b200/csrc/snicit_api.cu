// snicit_api.cu -- host runtime of libsnicit.so: the C ABI of include/snicit.h.
//
// Owns the device copies of the network, the per-batch workspace and the stream, validates every
// argument, and sequences the kernels of the hot path:
//   a1 pre-convergence layers (Eq. 1)  ->  a2 sampling + sum downsampling  ->  a3 Alg. 1 pruning
//   ->  a4 Alg. 2 mapping + residues  ->  a5 post-convergence layers (Eq. 5) + row compaction
//   ->  a6 Eq. 6 recovery + categories.
// No computation of the method happens on the host; host code only launches kernels, moves
// buffers the caller asked for, and reads device counters.
#include <cuda_runtime.h>
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <string>
#include <vector>

#include "../../include/snicit.h"
#include "snicit_internal.cuh"

using namespace snicit;

// the Python binding mirrors these structs (paper_conf_icpp_jiangh0h23_b200/_lib.py; tests/test_abi.py)
static_assert(sizeof(snicit_options) == 60, "snicit_options layout");
static_assert(sizeof(snicit_stats_t) == 200, "snicit_stats_t layout");

namespace {

thread_local std::string g_last_error;

snicit_status fail(snicit_status st, const std::string& msg) {
    g_last_error = msg;
    return st;
}

#define CUDA_TRY(expr)                                                                            \
    do {                                                                                          \
        cudaError_t _e = (expr);                                                                  \
        if (_e != cudaSuccess)                                                                    \
            return fail(_e == cudaErrorMemoryAllocation ? SNICIT_E_OOM : SNICIT_E_CUDA,          \
                        std::string(#expr) + ": " + cudaGetErrorString(_e));                     \
    } while (0)

template <typename T>
struct DevBuf {
    T* p = nullptr;
    size_t n = 0;
    cudaError_t ensure(size_t count) {
        if (count <= n && p) return cudaSuccess;
        if (p) cudaFree(p);
        p = nullptr;
        n = 0;
        cudaError_t e = cudaMalloc(&p, std::max<size_t>(count, 1) * sizeof(T));
        if (e == cudaSuccess) n = count;
        return e;
    }
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        n = 0;
    }
};

// Every entry point that touches the GPU switches to the handle's device and restores the caller's
// current device on return (the library never leaves the caller's device changed).
struct DeviceGuard {
    int prev = -1;
    cudaError_t status = cudaSuccess;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (dev >= 0) status = cudaSetDevice(dev);
    }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

// device pointers the kernels access with 16-byte vector / TMA bulk operations
inline bool misaligned16(const void* p) { return p && (reinterpret_cast<uintptr_t>(p) & 15u) != 0; }

// device counters (one int each)
enum Counter {
    CNT_LIVE0 = 0, CNT_LIVE1, CNT_LIVE2, CNT_ORD, CNT_RES0, CNT_RES1, CNT_NCENT, CNT_SEFF, CNT_ALL, CNT_NCAT,
    CNT_WORK, CNT_ALIVE, CNT_CDONE, CNT_PFWORK, CNT_PFCONST, CNT_CCOUNT, CNT_PROBE, CNT_NEED, CNT_N
};

}  // namespace

struct snicit_network {
    int device = 0;
    int N = 0, L = 0;
    float ymax = 32.f;
    int num_sms = 148;
    cudaStream_t stream = nullptr;
    std::vector<LayerPlan> plan;
    std::vector<uint8_t> dead_ok;  // dead_ok[l]: all biases of layers >= l are <= 0 (R23)
    bool idx16 = true;
    bool has_ell = true;  // ELL copies exist (CSC loads); compact circulant loads have none
    // weights
    DevBuf<uint16_t> idx16_d;
    DevBuf<int32_t> idx32_d;
    DevBuf<float> val_d;
    DevBuf<uint8_t> len_d;
    DevBuf<float> wtab_d;
    std::vector<float> wtab_h;  // host copy (weights passed as kernel parameters)
    // general-CSC row-interleaved kernel schedules (kernels_gen.cu), per layer with plan[l].gen
    int grl = 0;                  // outputs per warp instruction G (1 / 4 / 16), 0 = kernel unavailable
    DevBuf<uint16_t> gidx_d;
    DevBuf<float> gval_d;
    DevBuf<uint16_t> gsched_d;
    double gen_cost = 0.0;        // mean shared-memory wavefronts per tap of the schedules (1 = none lost)
    DevBuf<float> bias_d;
    DevBuf<PostLayer> post_layers_d;  // per-layer descriptors for the fused post-convergence kernels
    DevBuf<PreFusedLayer> pf_layers_d;  // per-layer descriptors of the row-resident pre-convergence kernel
    std::vector<PreFusedLayer> pf_layers_h;
    std::vector<uint8_t> pf_elig;       // layer l can run in the row-resident kernel
    DevBuf<unsigned long long> pf_full; // full-row layer evaluations of the last fused pre phase
    DevBuf<float> a_all;              // [(L - t)][s][N] centroid pre-activations (fused post mode)
    // workspace
    int64_t cap_rows = 0;
    int cap_s = 0, cap_n = 0;
    DevBuf<float> Ya, Yb;
    DevBuf<int> list0, list1, res0, res1, M, cslot, catlist, cent, col_idx, iota_s;
    DevBuf<uint8_t> flag_pos, live_row, ne_row, cat, ne_t;
    DevBuf<float> cbuf0, cbuf1, ac;
    DevBuf<int> cscratch;  // per-chunk counts of the ordered compaction
    DevBuf<uint8_t> segflag;  // row flags OR-ed by segmented layers (kept zero by the clearing compaction)
    DevBuf<int> rowctr;       // per-position warp counters of the column-streaming kernel (self-clearing)
    DevBuf<unsigned> cmin, cmax;  // constant-row mode: per position output range bits (self-restoring)
    DevBuf<int> clist, clayer;    // constant rows of the per-layer pre phase (R26)
    DevBuf<float> cval;
    DevBuf<int> cfrom;        // per centroid: first post layer with a constant a_c row (residual_traj)
    DevBuf<int> dist;         // [rows][s] L0 distances of Alg. 2 (map_residual pass 1)
    DevBuf<int> rnnz;         // [rows] non-zeros of each residue row at t
    DevBuf<int> need;         // [rows] list positions whose Alg. 2 distances are computed
    DevBuf<float> acs;        // [s][L - t] constant centroid pre-activations from cfrom on
    DevBuf<float2> wb_d;      // [L] (w0, b0) per layer (first bias of the layer)
    DevBuf<float> probe0, probe1;  // dynamic t: the probe rows (ping-pong)
    DevBuf<int> pstat;             // dynamic t: per probe layer (live, identical, distinct)
    DevBuf<unsigned long long> phash;  // dynamic t: per probe layer and row (hash, live)
    DevBuf<unsigned long long> dynbuf; // per-layer dynamics histograms (options.timing): pre [2][t + 1], post [2][L - t + 1]
    bool dyn_pre = false, dyn_post = false;
    int probe_layers = 0;
    DevBuf<uint8_t> rconst;   // rows constant at t (R26): flag + value, set by the pre phase
    DevBuf<float> rval;
    bool last_pre_const = false;
    DevBuf<uint32_t> bits;    // packed binary input rows (snicit_infer_packed, host bits)
    DevBuf<int> bits_ready;   // per chunk of uploaded rows: set by the copy engine after the chunk
    cudaStream_t copy_stream = nullptr;  // non-blocking upload stream (overlaps the row-resident kernel)
    cudaEvent_t cev[2] = {nullptr, nullptr};
    int* h_ones = nullptr;    // pinned source of the ready flags
    DevBuf<int> cdone;        // per centroid: carried to L by the constant-row kernel
    DevBuf<double> F;
    DevBuf<int> counters;
    int* h_counters = nullptr;  // pinned mirror
    // last-run state
    bool have_result = false;
    int64_t last_batch = 0, last_offset = 0;
    int last_t = 0;
    int last_s = 0, last_n = 0;
    bool last_converted = false;
    int live_counter = 0;  // which CNT_LIVE* holds the live count at t
    int res_final_counter = -1;  // counter holding the non-empty residue rows after the last layer
    bool last_fused = false;
    bool last_const = false;  // the constant-row centroid kernel ran in the last infer
    bool last_cluster = false;
    bool last_kernel_circ = false;
    bool last_pre_fused = false;
    bool last_dead_zeroed = false;  // the row-resident kernel wrote dead rows' zeros into y_out
    bool res_at_t_lazy = false;     // residual_at_t is read from CNT_RES0 by snicit_stats
    snicit_stats_t stats{};
    cudaEvent_t ev[10] = {};  // phase events [0..5]; map_residual [6, 7]; residue trajectories [8, 9]
    bool ev_map = false, ev_res = false;  // the kernel events of the last timed infer were recorded
    DevBuf<unsigned long long> ctr64;     // work counters of the last infer (Ctr64)
    std::vector<cudaEvent_t> lev;  // 2 per pre-convergence layer (timing == 2)
    DevBuf<int> hist;              // active rows at the start of each pre-convergence layer
    int prof_layers = 0;
};


// ---------------------------------------------------------------------------------------- load helpers
static snicit_status net_device_init(snicit_network* net, int cuda_device) {
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev < 1) return fail(SNICIT_E_CUDA, "no CUDA device");
    if (cuda_device < 0 || cuda_device >= ndev) return fail(SNICIT_E_INVALID_ARG, "bad cuda_device");
    cudaDeviceProp prop;
    cudaError_t pe = cudaGetDeviceProperties(&prop, cuda_device);
    if (pe != cudaSuccess) return fail(SNICIT_E_CUDA, cudaGetErrorString(pe));
    if (prop.major != 10)
        return fail(SNICIT_E_CUDA, "libsnicit is built for sm_100a (B200); device is sm_" +
                                       std::to_string(prop.major) + std::to_string(prop.minor));
    net->num_sms = prop.multiProcessorCount;
    net->device = cuda_device;
    cudaSetDevice(cuda_device);
    return SNICIT_OK;
}

// per-layer uniform-bias flag (SDGC: a constant per benchmark, Table 1) and dead_ok[l]: every bias
// of layers >= l is <= 0, so an all-zero row stays zero (R23)
static void net_bias_flags(snicit_network* net, const float* bias) {
    const int N = net->N, L = net->L;
    for (int l = 0; l < L; ++l) {
        bool ub = true;
        const float* b = bias + (int64_t)l * N;
        for (int j = 1; j < N && ub; ++j) ub = b[j] == b[0] && std::signbit(b[j]) == std::signbit(b[0]);
        net->plan[l].ubias = ub;
    }
    net->dead_ok.assign(L + 1, 1);
    for (int l = L - 1; l >= 0; --l) {
        bool ok = net->dead_ok[l + 1];
        for (int j = 0; j < N; ++j)
            if (bias[(int64_t)l * N + j] > 0.0f) ok = false;
        net->dead_ok[l] = ok ? 1 : 0;
    }
}

template <typename B, typename T>
static cudaError_t upload(B& buf, const T* host, size_t count) {
    cudaError_t e = buf.ensure(count);
    if (e != cudaSuccess) return e;
    if (count) return cudaMemcpy(buf.p, host, count * sizeof(T), cudaMemcpyHostToDevice);
    return cudaSuccess;
}

// weight table, bias, fused-post layer descriptors, counters, events (after the ELL arrays, if any)
static cudaError_t net_upload_common(snicit_network* net, const float* bias, const std::vector<float>& wtab) {
    const int N = net->N, L = net->L;
    net->wtab_h = wtab;
    cudaError_t e = upload(net->wtab_d, wtab.data(), wtab.size());
    if (e == cudaSuccess) e = upload(net->bias_d, bias, (size_t)L * N);
    if (e == cudaSuccess) {
        std::vector<PostLayer> pls(L);
        for (int l = 0; l < L; ++l) {
            const LayerPlan& pl = net->plan[l];
            PostLayer& d = pls[l];
            memset(&d, 0, sizeof(d));
            d.kind = pl.kind != 0 ? 1 : 0;
            d.cls = pl.kind != 0 ? circ_class_of(N, pl.nu) : 0;
            d.nu = pl.nu;
            d.K = pl.K;
            d.uniform_w = pl.uniform ? 1 : 0;
            d.ubias = pl.ubias ? 1 : 0;
            d.w0 = pl.w0;
            d.b0 = bias[(int64_t)l * N];
            d.bias = net->bias_d.p + (size_t)l * N;
            d.wtab = (pl.kind != 0 && !pl.uniform) ? net->wtab_d.p + pl.w_off : nullptr;
            if (net->has_ell) {
                d.idx16 = net->idx16 ? net->idx16_d.p + pl.ell_off : nullptr;
                d.idx32 = net->idx16 ? nullptr : net->idx32_d.p + pl.ell_off;
                d.val = pl.uniform ? nullptr : net->val_d.p + pl.ell_off;
                d.len = pl.ragged ? net->len_d.p + (size_t)l * N : nullptr;
            }
        }
        e = upload(net->post_layers_d, pls.data(), pls.size());
    }
    if (e == cudaSuccess) {
        // row-resident pre-convergence kernel (kernels_pre_fused.cu): circulant, 32 taps, uniform weight
        // and bias; stride classes nu == 1, Q == 32, or nu >= 32 with Q >= 64 and Q % 32 == 0
        net->pf_layers_h.assign(L, PreFusedLayer{});
        net->pf_elig.assign(L, 0);
        for (int l = 0; l < L; ++l) {
            const LayerPlan& pl = net->plan[l];
            PreFusedLayer& d = net->pf_layers_h[l];
            d.nu = pl.nu;
            d.w0 = pl.w0;
            d.b0 = bias[(int64_t)l * N];
            d.dead_next = net->dead_ok[l + 1];
            {  // constant row YMAX through this layer: the kernel's chain (acc = fma(v, w0, acc) x 32, + b0)
                float acc = 0.0f;
                for (int n = 0; n < 32; ++n) acc = std::fma(net->ymax, pl.w0, acc);
                const float z = acc + d.b0;
                d.ymax_fixed = std::fmin(std::fmax(z, 0.0f), net->ymax) == net->ymax ? 1 : 0;
            }
            d.cls = -1;
            if (pl.kind != 0 && pl.K == 32 && pl.uniform && pl.ubias && pl.nu >= 1 && N % pl.nu == 0) {
                const int Q = N / pl.nu;
                if (pl.nu == 1)
                    d.cls = PF_NU1;
                else if (Q == 32)
                    d.cls = PF_Q32;
                else if (pl.nu >= 32 && Q >= 64 && Q % 32 == 0)
                    d.cls = PF_STR;
            }
            net->pf_elig[l] = d.cls >= 0 ? 1 : 0;
        }
        e = upload(net->pf_layers_d, net->pf_layers_h.data(), net->pf_layers_h.size());
    }
    if (e == cudaSuccess) {
        std::vector<float2> wb(L);
        for (int l = 0; l < L; ++l) wb[l] = make_float2(net->plan[l].w0, bias[(int64_t)l * N]);
        e = upload(net->wb_d, wb.data(), wb.size());
    }
    if (e == cudaSuccess) e = net->pf_full.ensure(2);
    if (e == cudaSuccess) e = net->counters.ensure(CNT_N);
    if (e == cudaSuccess) e = cudaMallocHost(&net->h_counters, sizeof(int) * CNT_N);
    for (int i = 0; i < 10 && e == cudaSuccess; ++i) e = cudaEventCreate(&net->ev[i]);
    if (e == cudaSuccess) e = net->ctr64.ensure(C64_N);
    return e;
}

extern "C" {

void snicit_default_options(snicit_options* opt) {
    if (!opt) return;
    memset(opt, 0, sizeof(*opt));
    opt->n_segments = 16;
    opt->eta = 0.03f;
    opt->eps = 0.03f;
    opt->prune_eps = 0.0f;  // exact (R8)
    opt->drop_dead_rows = 1;
    opt->kernel = SNICIT_KERNEL_AUTO;
    opt->timing = 0;
    opt->ne_interval = 64;
    opt->post_mode = 0;
    opt->post_cluster = 1;
    opt->post_const = 1;
    opt->pre_fused = 1;
    opt->pre_const = 1;
    opt->res_sparse = 1;
    opt->dyn_t = 0;
}

const char* snicit_last_error(void) { return g_last_error.c_str(); }
int32_t snicit_abi_version(void) { return SNICIT_ABI_VERSION; }

void snicit_free_network(snicit_network* net) {
    if (!net) return;
    DeviceGuard dg(net->device);
    if (dg.status == cudaSuccess && net->stream) cudaStreamSynchronize(net->stream);
    net->idx16_d.release();
    net->idx32_d.release();
    net->val_d.release();
    net->len_d.release();
    net->wtab_d.release();
    net->gidx_d.release();
    net->gval_d.release();
    net->gsched_d.release();
    net->bias_d.release();
    net->Ya.release();
    net->Yb.release();
    for (auto* b : {&net->list0, &net->list1, &net->res0, &net->res1, &net->M, &net->cslot, &net->catlist, &net->cent,
                    &net->col_idx, &net->iota_s, &net->counters})
        b->release();
    for (auto* b : {&net->flag_pos, &net->live_row, &net->ne_row, &net->cat, &net->ne_t}) b->release();
    net->cbuf0.release();
    net->cbuf1.release();
    net->cscratch.release();
    net->segflag.release();
    net->rowctr.release();
    net->bits.release();
    net->cdone.release();
    net->ac.release();
    net->F.release();
    if (net->h_counters) cudaFreeHost(net->h_counters);
    if (net->h_ones) cudaFreeHost(net->h_ones);
    for (auto& e : net->cev)
        if (e) cudaEventDestroy(e);
    if (net->copy_stream) cudaStreamDestroy(net->copy_stream);
    net->bits_ready.release();
    for (auto& e : net->ev)
        if (e) cudaEventDestroy(e);
    for (auto& e : net->lev)
        if (e) cudaEventDestroy(e);
    net->hist.release();
    net->post_layers_d.release();
    net->pf_layers_d.release();
    net->pf_full.release();
    net->cmin.release();
    net->cmax.release();
    net->clist.release();
    net->clayer.release();
    net->cval.release();
    net->rconst.release();
    net->cfrom.release();
    net->rval.release();
    net->a_all.release();
    net->ctr64.release();
    net->dist.release();
    net->rnnz.release();
    net->need.release();
    net->acs.release();
    net->wb_d.release();
    net->probe0.release();
    net->probe1.release();
    net->pstat.release();
    net->phash.release();
    net->dynbuf.release();
    delete net;
}

snicit_status snicit_load_network(int32_t N, int32_t L, snicit_format fmt, const int64_t* ptr, const int32_t* idx,
                                  const float* val, const float* bias, float ymax, int32_t cuda_device,
                                  snicit_network** out) {
    if (!out) return fail(SNICIT_E_INVALID_ARG, "out is NULL");
    *out = nullptr;
    DeviceGuard dg(-1);  // net_device_init switches to cuda_device; the caller's device is restored
    if (N < 1 || L < 1) return fail(SNICIT_E_INVALID_ARG, "n_neurons and n_layers must be >= 1");
    if (!ptr || !bias) return fail(SNICIT_E_INVALID_ARG, "ptr/bias NULL");
    if (!(ymax > 0.0f) || std::isnan(ymax)) return fail(SNICIT_E_INVALID_ARG, "ymax must be > 0");
    if (fmt != SNICIT_CSC && fmt != SNICIT_CSR) return fail(SNICIT_E_INVALID_ARG, "bad format");
    if (N % 4 != 0) return fail(SNICIT_E_UNSUPPORTED, "n_neurons must be a multiple of 4 (16-byte rows)");
    // ---- host-side validation and conversion to per-layer column lists (stored order kept)
    std::vector<std::vector<int32_t>> cidx(N);
    std::vector<std::vector<float>> cval(N);
    const int64_t nnz_total = ptr[(int64_t)L * (N + 1) - 1];
    if (nnz_total < 0) return fail(SNICIT_E_BAD_SPARSE, "negative nnz");
    if (nnz_total > 0 && (!idx || !val)) return fail(SNICIT_E_INVALID_ARG, "idx/val NULL");
    for (int64_t i = 0; i < nnz_total; ++i)
        if (!std::isfinite(val[i])) return fail(SNICIT_E_INVALID_ARG, "non-finite weight");
    for (int64_t i = 0; i < (int64_t)L * N; ++i)
        if (!std::isfinite(bias[i])) return fail(SNICIT_E_INVALID_ARG, "non-finite bias");

    auto* net = new snicit_network();
    net->device = cuda_device;
    net->N = N;
    net->L = L;
    net->ymax = ymax;
    net->idx16 = N <= 65536;
    net->plan.resize(L);

    std::vector<int> Ks(L);
    size_t ell_total = 0;
    std::vector<std::vector<int32_t>> lay_idx(L);
    std::vector<std::vector<float>> lay_val(L);
    std::vector<std::vector<uint8_t>> lay_len(L);
    std::vector<float> wtab;
    std::vector<uint8_t> mark(N, 0);
    net->grl = gen_rows_per_tile(N);
    size_t gen_total = 0;
    int gen_layers = 0;
    double gen_cost_sum = 0.0;
    std::vector<uint16_t> g_idx;
    std::vector<float> g_val;
    std::vector<uint16_t> g_sched;
    for (int l = 0; l < L; ++l) {
        const int64_t* p = ptr + (int64_t)l * (N + 1);
        if (l > 0 && p[0] != ptr[(int64_t)l * (N + 1) - 1]) {
            snicit_free_network(net);
            return fail(SNICIT_E_BAD_SPARSE, "layer offsets not contiguous at layer " + std::to_string(l));
        }
        if (l == 0 && p[0] != 0) {
            snicit_free_network(net);
            return fail(SNICIT_E_BAD_SPARSE, "ptr[0] must be 0");
        }
        for (int j = 0; j < N; ++j) {
            cidx[j].clear();
            cval[j].clear();
        }
        for (int j = 0; j < N; ++j) {
            if (p[j + 1] < p[j]) {
                snicit_free_network(net);
                return fail(SNICIT_E_BAD_SPARSE, "ptr not monotone");
            }
            for (int64_t e = p[j]; e < p[j + 1]; ++e) {
                const int32_t k = idx[e];
                if (k < 0 || k >= N) {
                    snicit_free_network(net);
                    return fail(SNICIT_E_BAD_SPARSE, "index out of range");
                }
                if (fmt == SNICIT_CSC) {
                    cidx[j].push_back(k);
                    cval[j].push_back(val[e]);
                } else {  // CSR: entry (input j, output k); columns then ascending in input
                    cidx[k].push_back(j);
                    cval[k].push_back(val[e]);
                }
            }
        }
        int K = 0;
        bool ragged = false;
        for (int j = 0; j < N; ++j) {
            for (int32_t k : cidx[j]) {
                if (mark[k]) {
                    for (int32_t kk : cidx[j]) mark[kk] = 0;
                    snicit_free_network(net);
                    return fail(SNICIT_E_BAD_SPARSE, "duplicate index in a column of layer " + std::to_string(l));
                }
                mark[k] = 1;
            }
            for (int32_t k : cidx[j]) mark[k] = 0;
            K = std::max<int>(K, (int)cidx[j].size());
        }
        for (int j = 0; j < N; ++j)
            if ((int)cidx[j].size() != K) ragged = true;
        if (K > 255) {
            snicit_free_network(net);
            return fail(SNICIT_E_UNSUPPORTED, "more than 255 inputs per output neuron");
        }
        Ks[l] = K;
        LayerPlan& pl = net->plan[l];
        pl.K = K;
        pl.ragged = ragged;
        pl.ell_off = ell_total;
        ell_total += (size_t)K * N;
        // uniform value?
        bool uniform = true;
        float w0 = 0.f;
        bool first = true;
        for (int j = 0; j < N && uniform; ++j)
            for (float v : cval[j]) {
                if (first) {
                    w0 = v;
                    first = false;
                } else if (v != w0 || std::signbit(v) != std::signbit(w0)) {
                    uniform = false;
                    break;
                }
            }
        pl.uniform = uniform;
        pl.w0 = w0;
        // circulant? column j = (j + n*nu) mod N for n = 0..K-1, per-n weights uniform over j
        pl.kind = 0;
        pl.nu = 0;
        if (!ragged && K >= 2) {
            const int nu = (int)(((int64_t)cidx[0][1] - cidx[0][0] + N) % N);
            bool circ = cidx[0][0] == 0 && (circ_supported(N, K, nu) || circ_seg_supported(N, K, nu));
            for (int j = 0; j < N && circ; ++j)
                for (int n = 0; n < K; ++n) {
                    if (cidx[j][n] != (int32_t)(((int64_t)j + (int64_t)n * nu) % N) || cval[j][n] != cval[0][n] ||
                        std::signbit(cval[j][n]) != std::signbit(cval[0][n])) {
                        circ = false;
                        break;
                    }
                }
            if (circ) {
                pl.kind = circ_supported(N, K, nu) ? 1 : 2;  // whole rows staged, or segmented rows
                pl.col = circ_col_supported(N, K, nu);
                pl.nu = nu;
                pl.w_off = wtab.size();
                for (int n = 0; n < K; ++n) wtab.push_back(cval[0][n]);
            }
        }
        // ELL (n-major) copy for every layer (ELL kernel and debug comparisons)
        lay_idx[l].assign((size_t)K * N, 0);
        lay_val[l].assign((size_t)K * N, 0.0f);
        if (ragged) lay_len[l].assign(N, 0);
        for (int j = 0; j < N; ++j) {
            for (size_t n = 0; n < cidx[j].size(); ++n) {
                lay_idx[l][n * N + j] = cidx[j][n];
                lay_val[l][n * N + j] = cval[j][n];
            }
            if (ragged) lay_len[l][j] = (uint8_t)cidx[j].size();
        }
        // general-CSC kernel schedule: every non-circulant layer; circulant layers too while the arrays stay
        // small (SNICIT_KERNEL_ELL runs them through the same kernel in tests)
        pl.gen = false;
        if (net->grl > 0 && (pl.kind == 0 || (size_t)L * N * 32 <= ((size_t)16 << 20))) {
            pl.gen = true;
            pl.gkp = (K + 3) & ~3;
            if (pl.gkp == 0) pl.gkp = 4;
            pl.gen_off = gen_total;
            gen_total += (size_t)N * ((pl.gkp + 7) & ~7);
            g_idx.resize(gen_total);
            if (!pl.uniform) g_val.resize(gen_total);
            if (net->grl == 16) g_sched.resize((size_t)(gen_layers + 1) * N);
            uint16_t* sch = net->grl == 16 ? g_sched.data() + (size_t)gen_layers * N : nullptr;
            gen_cost_sum += gen_build_layer(N, net->grl, pl.gkp, cidx, cval, g_idx.data() + pl.gen_off,
                                            pl.uniform ? nullptr : g_val.data() + pl.gen_off, sch);
            ++gen_layers;
        }
    }
    net_bias_flags(net, bias);
    // ---- device (validation above needs no GPU, so bad input is reported on any host)
    {
        const snicit_status ds = net_device_init(net, cuda_device);
        if (ds != SNICIT_OK) {
            const std::string msg = g_last_error;
            snicit_free_network(net);
            return fail(ds, msg);
        }
    }
    // ---- upload
    auto up = [&](auto& buf, const auto* host, size_t count) -> cudaError_t {
        cudaError_t e = buf.ensure(count);
        if (e != cudaSuccess) return e;
        if (count) return cudaMemcpy(buf.p, host, count * sizeof(*host), cudaMemcpyHostToDevice);
        return cudaSuccess;
    };
    cudaError_t e = cudaSuccess;
    {
        std::vector<float> allv(ell_total);
        for (int l = 0; l < L; ++l) std::copy(lay_val[l].begin(), lay_val[l].end(), allv.begin() + net->plan[l].ell_off);
        if (net->idx16) {
            std::vector<uint16_t> alli(ell_total);
            for (int l = 0; l < L; ++l)
                for (size_t i = 0; i < lay_idx[l].size(); ++i) alli[net->plan[l].ell_off + i] = (uint16_t)lay_idx[l][i];
            e = up(net->idx16_d, alli.data(), ell_total);
        } else {
            std::vector<int32_t> alli(ell_total);
            for (int l = 0; l < L; ++l) std::copy(lay_idx[l].begin(), lay_idx[l].end(), alli.begin() + net->plan[l].ell_off);
            e = up(net->idx32_d, alli.data(), ell_total);
        }
        if (e == cudaSuccess) e = up(net->val_d, allv.data(), ell_total);
        bool any_rag = false;
        for (int l = 0; l < L; ++l) any_rag |= net->plan[l].ragged;
        if (e == cudaSuccess && any_rag) {
            std::vector<uint8_t> alll((size_t)L * N, 0);
            for (int l = 0; l < L; ++l)
                if (net->plan[l].ragged) std::copy(lay_len[l].begin(), lay_len[l].end(), alll.begin() + (size_t)l * N);
            e = up(net->len_d, alll.data(), alll.size());
        }
    }
    if (e == cudaSuccess && gen_layers > 0) {
        net->gen_cost = gen_cost_sum / gen_layers;
        // weights of non-uniform layers: fill uniform layers' ranges too (one array for all layers)
        if (!g_val.empty()) g_val.resize(gen_total, 0.0f);
        e = up(net->gidx_d, g_idx.data(), gen_total);
        if (e == cudaSuccess && !g_val.empty()) e = up(net->gval_d, g_val.data(), gen_total);
        if (e == cudaSuccess && !g_sched.empty()) e = up(net->gsched_d, g_sched.data(), g_sched.size());
        // per-layer schedule slot (sched arrays are indexed by the order of gen layers)
        int gi = 0;
        for (int l = 0; l < L; ++l)
            if (net->plan[l].gen) net->plan[l].gsched_idx = gi++;
    }
    if (e == cudaSuccess) e = net_upload_common(net, bias, wtab);
    if (e != cudaSuccess) {
        snicit_free_network(net);
        return fail(e == cudaErrorMemoryAllocation ? SNICIT_E_OOM : SNICIT_E_CUDA, cudaGetErrorString(e));
    }
    *out = net;
    return SNICIT_OK;
}

snicit_status snicit_load_network_circulant(int32_t N, int32_t L, const int32_t* nu, int32_t K, const float* w,
                                            const float* bias, float ymax, int32_t cuda_device,
                                            snicit_network** out) {
    if (!out) return fail(SNICIT_E_INVALID_ARG, "out is NULL");
    *out = nullptr;
    DeviceGuard dg(-1);
    if (N < 1 || L < 1 || K < 1) return fail(SNICIT_E_INVALID_ARG, "n_neurons, n_layers, K must be >= 1");
    if (!nu || !w || !bias) return fail(SNICIT_E_INVALID_ARG, "nu/w/bias NULL");
    if (!(ymax > 0.0f) || std::isnan(ymax)) return fail(SNICIT_E_INVALID_ARG, "ymax must be > 0");
    if (N % 4 != 0) return fail(SNICIT_E_UNSUPPORTED, "n_neurons must be a multiple of 4 (16-byte rows)");
    for (int64_t i = 0; i < (int64_t)L * K; ++i)
        if (!std::isfinite(w[i])) return fail(SNICIT_E_INVALID_ARG, "non-finite weight");
    for (int64_t i = 0; i < (int64_t)L * N; ++i)
        if (!std::isfinite(bias[i])) return fail(SNICIT_E_INVALID_ARG, "non-finite bias");
    auto* net = new snicit_network();
    net->N = N;
    net->L = L;
    net->ymax = ymax;
    net->idx16 = N <= 65536;
    net->has_ell = false;
    net->plan.resize(L);
    std::vector<float> wtab;
    for (int l = 0; l < L; ++l) {
        const int v = nu[l];
        if (v < 1 || v > N || N % v != 0 || (int64_t)K * v > N) {
            snicit_free_network(net);
            return fail(SNICIT_E_BAD_SPARSE, "layer " + std::to_string(l) + ": stride must divide N with K*nu <= N");
        }
        if (!(circ_supported(N, K, v) || circ_seg_supported(N, K, v))) {
            snicit_free_network(net);
            return fail(SNICIT_E_UNSUPPORTED, "layer " + std::to_string(l) + ": no circulant kernel for (N, K, nu)");
        }
        LayerPlan& pl = net->plan[l];
        pl.kind = circ_supported(N, K, v) ? 1 : 2;
        pl.col = circ_col_supported(N, K, v);
        pl.nu = v;
        pl.K = K;
        pl.ragged = false;
        const float* wl = w + (int64_t)l * K;
        bool uniform = true;
        for (int n = 1; n < K; ++n) uniform &= wl[n] == wl[0] && std::signbit(wl[n]) == std::signbit(wl[0]);
        pl.uniform = uniform;
        pl.w0 = wl[0];
        pl.w_off = wtab.size();
        for (int n = 0; n < K; ++n) wtab.push_back(wl[n]);
        pl.ell_off = 0;
    }
    net_bias_flags(net, bias);
    snicit_status ds = net_device_init(net, cuda_device);
    if (ds != SNICIT_OK) {
        const std::string msg = g_last_error;
        snicit_free_network(net);
        return fail(ds, msg);
    }
    cudaError_t e = net_upload_common(net, bias, wtab);
    if (e != cudaSuccess) {
        snicit_free_network(net);
        return fail(e == cudaErrorMemoryAllocation ? SNICIT_E_OOM : SNICIT_E_CUDA, cudaGetErrorString(e));
    }
    *out = net;
    return SNICIT_OK;
}

snicit_status snicit_set_stream(snicit_network* net, void* s) {
    if (!net) return fail(SNICIT_E_INVALID_ARG, "net NULL");
    net->stream = (cudaStream_t)s;
    return SNICIT_OK;
}

int32_t snicit_debug_range_tables(float w0, float b0, float ymax, int32_t kmax, float* hi, float* lo) {
    if (!hi || !lo || kmax < 1 || kmax > kRangeK || !(ymax > 0.0f)) return SNICIT_E_INVALID_ARG;
    PreFusedLayer d{};
    d.w0 = w0;
    d.b0 = b0;
    float h[kRangeK], l_[kRangeK];
    const bool ok = range_tables(&d, 1, ymax, h, l_);
    for (int k = 0; k < kmax; ++k) {
        hi[k] = ok ? h[k] : INFINITY;
        lo[k] = ok ? l_[k] : -1.0f;
    }
    return ok ? 1 : 0;
}

snicit_status snicit_debug_gen_schedule(int32_t N, int32_t K, const int32_t* cols, int32_t* rows_per_tile,
                                        double* cost) {
    if (N < 1 || K < 1 || K > 255 || !cols || !rows_per_tile || !cost)
        return fail(SNICIT_E_INVALID_ARG, "bad arguments");
    std::vector<std::vector<int32_t>> cidx(N);
    std::vector<std::vector<float>> cval(N);
    for (int j = 0; j < N; ++j)
        for (int n = 0; n < K; ++n) {
            const int32_t k = cols[(size_t)j * K + n];
            if (k < 0 || k >= N) return fail(SNICIT_E_INVALID_ARG, "index out of range");
            cidx[j].push_back(k);
            cval[j].push_back(1.0f);
        }
    const int rl = gen_rows_per_tile(N);
    *rows_per_tile = rl;
    *cost = 0.0;
    if (rl == 0) return SNICIT_OK;
    const int kp = (K + 3) & ~3;
    std::vector<uint16_t> idx((size_t)N * ((kp + 7) & ~7));
    std::vector<uint16_t> sched(N);
    *cost = gen_build_layer(N, rl, kp, cidx, cval, idx.data(), nullptr, sched.data());
    return SNICIT_OK;
}

int32_t snicit_layer_is_circulant(const snicit_network* net, int32_t l) {
    if (!net || l < 0 || l >= net->L) return -1;
    return net->plan[l].kind != 0 ? 1 : 0;
}

}  // extern "C"

// ---------------------------------------------------------------------------------------- helpers
static LayerArgs layer_args(snicit_network* net, int l, bool force_ell) {
    const LayerPlan& pl = net->plan[l];
    LayerArgs a{};
    a.thr_hi = INFINITY;  // range prediction (R30) off unless the constant-row pre path turns it on
    a.thr_lo = -1.0f;
    a.N = net->N;
    a.bias = net->bias_d.p + (size_t)l * net->N;
    a.ymax = net->ymax;
    a.K = pl.K;
    if (net->has_ell) {
        if (net->idx16)
            a.idx16 = net->idx16_d.p + pl.ell_off;
        else
            a.idx32 = net->idx32_d.p + pl.ell_off;
        a.val = pl.uniform ? nullptr : net->val_d.p + pl.ell_off;
        a.len = pl.ragged ? net->len_d.p + (size_t)l * net->N : nullptr;
    }
    if (pl.gen && net->grl > 0) {
        a.gidx = net->gidx_d.p + pl.gen_off;
        a.gval = pl.uniform ? nullptr : net->gval_d.p + pl.gen_off;
        a.gsched = net->grl == 16 ? net->gsched_d.p + (size_t)pl.gsched_idx * net->N : nullptr;
        a.grl = net->grl;
        a.gkp = pl.gkp;
    }
    a.w0 = pl.w0;
    a.uniform_bias = pl.ubias ? 1 : 0;
    if (pl.kind != 0 && !force_ell) {
        a.nu = pl.nu;
        a.wtab = pl.uniform ? nullptr : net->wtab_d.p + pl.w_off;
        a.wtab_host = pl.uniform ? nullptr : net->wtab_h.data() + pl.w_off;
    }
    return a;
}

static bool use_circ(const snicit_network* net, int l, int kernel_opt) {
    if (kernel_opt == SNICIT_KERNEL_ELL) return false;
    return net->plan[l].kind != 0;
}
// segmented circulant layers: a row spans several CTAs, so row flags are OR-ed into `segflag` and
// compacted by a separate (ordered, clearing) compaction instead of the fused append
static bool use_seg(const snicit_network* net, int l, int kernel_opt) {
    return use_circ(net, l, kernel_opt) && net->plan[l].kind == 2;
}
// strided circulant layers in PLAIN mode: the column-streaming kernel (rows from global memory, row
// flags OR-ed like the segmented kernel) unless SNICIT_KERNEL_CIRC_SMEM asks for the staged kernels
static bool use_col(const snicit_network* net, int l, int kernel_opt) {
    return use_circ(net, l, kernel_opt) && kernel_opt != SNICIT_KERNEL_CIRC_SMEM && net->plan[l].col;
}

// a general (ELL) layer on which a constant row stays constant: one weight, one bias, 32 entries in every
// column (the chain every output evaluates is the same, R26); the ELL kernels report row output ranges
static bool ell_const_ok(const snicit_network* net, int l, int kernel_opt) {
    const LayerPlan& pl = net->plan[l];
    return !use_circ(net, l, kernel_opt) && net->has_ell && pl.uniform && pl.ubias && !pl.ragged && pl.K == 32;
}

static cudaError_t run_layer(snicit_network* net, int l, int kernel_opt, int mode, LayerArgs a, int max_rows) {
    if (mode == MODE_PLAIN && use_col(net, l, kernel_opt))
        return launch_layer_circ_col(a, max_rows, net->num_sms, net->stream);
    if (use_seg(net, l, kernel_opt)) return launch_layer_circ_seg(a, mode, max_rows, net->num_sms, net->stream);
    if (use_circ(net, l, kernel_opt)) return launch_layer_circ(a, mode, max_rows, net->num_sms, net->stream);
    return launch_layer_ell(a, mode, max_rows, net->num_sms, net->stream);
}

static cudaError_t ensure_workspace(snicit_network* net, int64_t R, int s, int n) {
    const size_t rows = (size_t)std::max<int64_t>(R, 1);
    const size_t rn = rows * (size_t)net->N;
    cudaError_t e;
    if ((e = net->Ya.ensure(rn)) != cudaSuccess) return e;
    if ((e = net->Yb.ensure(rn)) != cudaSuccess) return e;
    for (auto* b : {&net->list0, &net->list1, &net->res0, &net->res1, &net->M, &net->cslot, &net->catlist})
        if ((e = b->ensure(rows)) != cudaSuccess) return e;
    for (auto* b : {&net->flag_pos, &net->live_row, &net->ne_row, &net->cat, &net->ne_t})
        if ((e = b->ensure(rows)) != cudaSuccess) return e;
    const size_t ss = (size_t)std::max(s, 1);
    for (auto* b : {&net->cbuf0, &net->cbuf1, &net->ac})
        if ((e = b->ensure(ss * net->N)) != cudaSuccess) return e;
    if ((e = net->cent.ensure(ss)) != cudaSuccess) return e;
    if ((e = net->col_idx.ensure(ss)) != cudaSuccess) return e;
    if ((e = net->iota_s.ensure(ss)) != cudaSuccess) return e;
    if ((e = net->F.ensure((size_t)std::max(n, 1) * ss)) != cudaSuccess) return e;
    if ((e = net->dist.ensure(rows * ss)) != cudaSuccess) return e;
    if ((e = net->rnnz.ensure(rows)) != cudaSuccess) return e;
    if ((e = net->need.ensure(rows)) != cudaSuccess) return e;
    if ((e = net->cscratch.ensure((size_t)compact_scratch_ints((int)rows))) != cudaSuccess) return e;
    if (net->segflag.n < rows) {
        if ((e = net->segflag.ensure(rows)) != cudaSuccess) return e;
        if ((e = cudaMemsetAsync(net->segflag.p, 0, rows, net->stream)) != cudaSuccess) return e;
    }
    if (net->cmin.n < rows) {
        if ((e = net->cmin.ensure(rows)) != cudaSuccess) return e;
        if ((e = cudaMemsetAsync(net->cmin.p, 0xff, rows * sizeof(unsigned), net->stream)) != cudaSuccess) return e;
    }
    if (net->cmax.n < rows) {
        if ((e = net->cmax.ensure(rows)) != cudaSuccess) return e;
        if ((e = cudaMemsetAsync(net->cmax.p, 0, rows * sizeof(unsigned), net->stream)) != cudaSuccess) return e;
    }
    for (auto* b : {&net->clist, &net->clayer})
        if ((e = b->ensure(rows)) != cudaSuccess) return e;
    if ((e = net->cval.ensure(rows)) != cudaSuccess) return e;
    if ((e = net->rconst.ensure(rows)) != cudaSuccess) return e;
    if ((e = net->rval.ensure(rows)) != cudaSuccess) return e;
    if (net->rowctr.n < rows) {
        if ((e = net->rowctr.ensure(rows)) != cudaSuccess) return e;
        if ((e = cudaMemsetAsync(net->rowctr.p, 0, rows * sizeof(int), net->stream)) != cudaSuccess) return e;
    }
    return cudaSuccess;
}

static cudaError_t read_counter(snicit_network* net, int which, int* outv) {
    cudaError_t e = cudaMemcpyAsync(net->h_counters + which, net->counters.p + which, sizeof(int),
                                    cudaMemcpyDeviceToHost, net->stream);
    if (e != cudaSuccess) return e;
    e = cudaStreamSynchronize(net->stream);
    if (e != cudaSuccess) return e;
    *outv = net->h_counters[which];
    return cudaSuccess;
}

extern "C" {

// Row-resident pre phase applicable?  (kernels_pre_fused.cu: circulant layers < t with 32 taps,
// uniform weight and bias, N / 32 in 32..512, t <= kPfMaxLayers, smem fits); *H = circular halo
// *cluster: the row is split over a thread-block cluster (kernels_pre_cluster.cu: N = 16384 / 32768 /
// 65536, every layer's stride supported): the default for rows a single CTA cannot hold (N > 16384; C4
// 31.8 -> 29.3 ms with R30 / R31 in the cluster kernel, round 2 (r02c)), on request (pre_fused = 4) at N = 16384,
// where the single-CTA kernel is faster;
// *bits_ok: packed input rows can be read by the chosen kernel
static bool pf_plan(const snicit_network* net, int tt, const snicit_options& opt, int R, int* H, int* gen,
                    bool* cluster = nullptr, bool* bits_ok = nullptr) {
    const int N = net->N;
    if (cluster) *cluster = false;
    if (bits_ok) *bits_ok = true;
    const bool base_ok = opt.pre_fused != 0 && tt > 0 && tt <= kPfMaxLayers && R > 0 && opt.kernel == SNICIT_KERNEL_AUTO;
    const bool want_cluster = opt.pre_fused == 4 || (opt.pre_fused == 1 && N > 16384);
    if (base_ok && want_cluster && pre_cluster_supported(N)) {
        bool ok = true;
        for (int l = 0; l < tt && ok; ++l) ok = net->pf_elig[l] != 0 && pre_cluster_class(N, net->plan[l].nu) >= 0;
        if (ok) {
            if (cluster) *cluster = true;
            if (bits_ok) *bits_ok = N % 128 == 0 && pre_cluster_class(N, net->plan[0].nu) <= 1;  // W partition at layer 0
            *H = 0;
            *gen = 0;
            return true;
        }
    }
    bool pf = base_ok && opt.pre_fused != 4 && pre_fused_threads(N) > 0;
    for (int l = 0; l < tt && pf; ++l) pf = net->pf_elig[l] != 0;
    int h = 96, g = 0;  // nu == 1 windows read 47 past an item, head items write 68; STR 31*nu
    if (pf) {
        for (int l = 0; l < tt; ++l)
            if (net->pf_layers_h[l].cls == PF_STR) {
                if (pre_fused_str_halo(N)) h = std::max(h, 31 * net->pf_layers_h[l].nu);
                if (net->pf_layers_h[l].nu != 32) g = 1;
            }
        h = (h + 31) / 32 * 32;
        if (opt.pre_fused != 5) {  // the split-layout kernel (kernels_pre_fused.cu)
            if (h > N || pre_fused_smem(N, h) > (size_t)227 * 1024) pf = false;
        } else {  // the paired-half layout (kernels_pre_pair.cu), on request
            const int hp = pre_pair_halo(N, net->pf_layers_h.data(), tt);
            if (hp < 0 || pre_pair_smem(N, hp) > (size_t)227 * 1024) pf = false;
        }
    }
    *H = h;
    *gen = g;
    return pf;
}

// Streamed upload of R host rows of `row_bytes` each into the device buffer `dst`: the copy engine
// delivers geometric chunks of rows (chunk c = rows [b (2^c - 1), b (2^(c+1) - 1)), b = kChunk0) on a
// side stream, each followed by its ready flag, while the row-resident kernel runs (it polls the flag
// of a row's chunk before loading the row), so the upload overlaps the compute.  The first rows
// arrive within microseconds and the whole batch takes a handful of API calls.  The handle's stream
// must wait on net->cev[1] before anything later reuses `dst` or the flags.
static cudaError_t stream_upload(snicit_network* net, void* dst, const void* src, size_t row_bytes, int R,
                                 const int** ready, int* ready_rows) {
    constexpr int kChunk0 = 512;
    int nch = 0;
    while ((long long)kChunk0 * ((1LL << nch) - 1) < R) ++nch;
    cudaError_t e;
    if (!net->copy_stream && (e = cudaStreamCreateWithFlags(&net->copy_stream, cudaStreamNonBlocking)) != cudaSuccess)
        return e;
    for (auto& ev : net->cev)
        if (!ev && (e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming)) != cudaSuccess) return e;
    if (!net->h_ones) {
        if ((e = cudaMallocHost(&net->h_ones, sizeof(int))) != cudaSuccess) return e;
        *net->h_ones = 1;
    }
    if ((e = net->bits_ready.ensure((size_t)std::max(nch, 1))) != cudaSuccess) return e;
    if ((e = cudaMemsetAsync(net->bits_ready.p, 0, sizeof(int) * std::max(nch, 1), net->stream)) != cudaSuccess) return e;
    if ((e = cudaEventRecord(net->cev[0], net->stream)) != cudaSuccess) return e;
    if ((e = cudaStreamWaitEvent(net->copy_stream, net->cev[0], 0)) != cudaSuccess) return e;
    for (int c = 0; c < nch; ++c) {
        const size_t r0 = (size_t)kChunk0 * ((1ull << c) - 1);
        const size_t nr = std::min<size_t>((size_t)kChunk0 << c, R - r0);
        if ((e = cudaMemcpyAsync(static_cast<char*>(dst) + r0 * row_bytes, static_cast<const char*>(src) + r0 * row_bytes,
                                 row_bytes * nr, cudaMemcpyHostToDevice, net->copy_stream)) != cudaSuccess)
            return e;
        if ((e = cudaMemcpyAsync(net->bits_ready.p + c, net->h_ones, sizeof(int), cudaMemcpyHostToDevice,
                                 net->copy_stream)) != cudaSuccess)
            return e;
    }
    if ((e = cudaEventRecord(net->cev[1], net->copy_stream)) != cudaSuccess) return e;
    *ready = net->bits_ready.p;
    *ready_rows = kChunk0;
    return cudaSuccess;
}

// Dynamic threshold layer ("determine t dynamically" is the paper's future work,
// P:1619-1621).  Any t gives the plain result, so t only decides the cost.  The first
// S = min(s, R) rows of the batch -- the rows Alg. 1 samples -- are run through the layers on
// the side; l* is the first layer after which every live probe row is identical (the clustering would find
// one centroid and no residue among them).  The rest of the batch converges later than its first rows
// do on average, and a late t is cheap (rows that became constant cost a scalar per layer, R26) while an
// early t leaves residue rows for hundreds of layers, so t = min(2 l*, tmax) (measured on C1/C2/C3:
// profiles/r02_dyn_t.md).  If the probe rows never become identical and more than S/2 of them are still
// distinct at tmax, clustering cannot compress the batch: the uncompressed path (t = L).
// Rows of N <= 24576: one kernel carries each probe row through all tmax layers and records per-layer
// hashes (one launch, one read-back); larger rows: per-layer launches, statistics read every 4 layers.
static cudaError_t choose_t(snicit_network* net, const float* src, const uint32_t* bits, float one, int R, int s,
                            int tmax, int* t_out) {
    const int N = net->N, L = net->L;
    const int S = std::min(std::min(s, R), 1024);
    cudaStream_t st = net->stream;
    cudaError_t e;
    if ((e = net->probe0.ensure((size_t)S * N)) != cudaSuccess) return e;
    if ((e = net->probe1.ensure((size_t)S * N)) != cudaSuccess) return e;
    if ((e = net->pstat.ensure((size_t)3 * (tmax + 1))) != cudaSuccess) return e;
    if ((e = net->iota_s.ensure((size_t)std::max(S, 1))) != cudaSuccess) return e;
    if (src)
        e = cudaMemcpyAsync(net->probe0.p, src, sizeof(float) * (size_t)S * N, cudaMemcpyDeviceToDevice, st);
    else
        e = launch_unpack_bits(bits, S, N, one, net->probe0.p, net->num_sms, st);
    if (e != cudaSuccess) return e;
    if ((e = launch_iota(net->iota_s.p, S, net->counters.p + CNT_PROBE, st)) != cudaSuccess) return e;
    if (N <= post_fused_max_n()) {  // one launch: probe rows through all tmax layers, per-layer hashes
        if ((e = net->phash.ensure((size_t)2 * tmax * S)) != cudaSuccess) return e;
        PostArgs pa{};
        pa.N = N;
        pa.L = L;
        pa.t = 0;
        pa.ymax = net->ymax;
        pa.layers = net->post_layers_d.p;
        if ((e = launch_probe_traj(pa, net->probe0.p, S, tmax, net->phash.p, st)) != cudaSuccess) return e;
        std::vector<unsigned long long> hv((size_t)2 * tmax * S);
        if ((e = cudaMemcpyAsync(hv.data(), net->phash.p, sizeof(unsigned long long) * hv.size(),
                                 cudaMemcpyDeviceToHost, st)) != cudaSuccess)
            return e;
        if ((e = cudaStreamSynchronize(st)) != cudaSuccess) return e;
        net->probe_layers = 1;
        int lstar = -1;
        for (int l = 0; l < tmax && lstar < 0; ++l) {
            bool have = false, ident = true;
            unsigned long long h0 = 0;
            for (int b = 0; b < S; ++b) {
                const unsigned long long hb = hv[2 * ((size_t)l * S + b)], live = hv[2 * ((size_t)l * S + b) + 1];
                if (!live) continue;
                if (!have) {
                    have = true;
                    h0 = hb;
                } else if (hb != h0) {
                    ident = false;
                }
            }
            if (!have || ident) lstar = l + 1;
        }
        if (lstar > 0) {
            *t_out = std::min(2 * lstar, tmax);
        } else {  // distinct live probe rows after layer tmax
            std::vector<unsigned long long> hs;
            for (int b = 0; b < S; ++b)
                if (hv[2 * ((size_t)(tmax - 1) * S + b) + 1]) hs.push_back(hv[2 * ((size_t)(tmax - 1) * S + b)]);
            std::sort(hs.begin(), hs.end());
            const int uniq = (int)(std::unique(hs.begin(), hs.end()) - hs.begin());
            *t_out = 2 * uniq > S ? L : tmax;
        }
        return cudaSuccess;
    }
    std::vector<int> h((size_t)3 * (tmax + 1));
    float* pin = net->probe0.p;
    float* pout = net->probe1.p;
    int done = 0, chosen = -1;
    net->probe_layers = 0;
    for (int l = 0; l < tmax && chosen < 0; ++l) {
        LayerArgs a = layer_args(net, l, false);
        a.yin = pin;
        a.yout = pout;
        a.rows = net->iota_s.p;
        a.count = net->counters.p + CNT_PROBE;
        a.row_ctr = net->rowctr.p;
        if ((e = run_layer(net, l, SNICIT_KERNEL_AUTO, MODE_PLAIN, a, S)) != cudaSuccess) return e;
        if ((e = launch_probe_stat(pout, S, N, net->pstat.p + 3 * (l + 1), st)) != cudaSuccess) return e;
        std::swap(pin, pout);
        net->probe_layers = l + 1;
        if ((l + 1) % 4 == 0 || l + 1 == tmax) {
            if ((e = cudaMemcpyAsync(h.data() + 3 * (done + 1), net->pstat.p + 3 * (done + 1),
                                     sizeof(int) * 3 * (l + 1 - done), cudaMemcpyDeviceToHost, st)) != cudaSuccess)
                return e;
            if ((e = cudaStreamSynchronize(st)) != cudaSuccess) return e;
            for (int k = done + 1; k <= l + 1 && chosen < 0; ++k)
                if (h[3 * k] == 0 || h[3 * k + 1]) chosen = std::min(2 * k, tmax);
            done = l + 1;
        }
    }
    if (chosen < 0) chosen = (2 * h[3 * tmax + 2] > S) ? L : tmax;
    *t_out = chosen;
    return cudaSuccess;
}

// y0_mode: 0 = y0 is a device pointer, 1 = host pointer, 2 = the input rows are already in net->Ya,
// 3 = packed binary rows `bits` (device-accessible, possibly host-mapped) read by the row-resident
// kernel (the caller checked pf_plan)
// (snicit_infer_packed unpacked them there)
static snicit_status infer_core(snicit_network* net, const float* y0, int64_t batch, int32_t y0_mode,
                                int64_t row_offset, int32_t t, int32_t s, const snicit_options* opt_in, float* y_out,
                                int32_t y_out_on_device, const uint32_t* bits = nullptr, float one = 1.0f,
                                const int* bits_ready = nullptr, int ready_rows = 0) {
    // (bits_ready / ready_rows: the ready flags of a streamed upload, set here for host fp32 rows)
    const int32_t y0_on_device = y0_mode == 0;
    if (!net) return fail(SNICIT_E_INVALID_ARG, "net NULL");
    if (batch < 0 || batch > 0x7fffffffLL) return fail(SNICIT_E_INVALID_ARG, "batch out of range");
    if (batch > 0 && !y0 && y0_mode < 2) return fail(SNICIT_E_INVALID_ARG, "y0 NULL");
    if (t < 0) return fail(SNICIT_E_INVALID_ARG, "threshold_layer < 0");
    if (s < 1) return fail(SNICIT_E_INVALID_ARG, "centroid_count < 1");
    if (s > 1024) return fail(SNICIT_E_UNSUPPORTED, "centroid_count > 1024");
    if (row_offset < 0) return fail(SNICIT_E_INVALID_ARG, "row_offset < 0");
    if ((y0_on_device && misaligned16(y0)) || (y_out_on_device && misaligned16(y_out)) ||
        (y0_mode == 3 && misaligned16(bits)))
        return fail(SNICIT_E_INVALID_ARG, "device y0 / y_out / bits must be 16-byte aligned");
    snicit_options opt;
    if (opt_in)
        opt = *opt_in;
    else
        snicit_default_options(&opt);
    if (opt.n_segments < 0 || opt.n_segments > net->N) return fail(SNICIT_E_INVALID_ARG, "n_segments out of range");
    if (!(opt.eps >= 0.0f) || std::isnan(opt.eta) || !(opt.prune_eps >= 0.0f))
        return fail(SNICIT_E_INVALID_ARG, "bad eta/eps/prune_eps");
    if (opt.kernel < 0 || opt.kernel > SNICIT_KERNEL_CIRC_SMEM) return fail(SNICIT_E_INVALID_ARG, "bad kernel option");
    if (opt.post_mode < 0 || opt.post_mode > 1) return fail(SNICIT_E_INVALID_ARG, "bad post_mode");
    if (opt.pre_fused < 0 || opt.pre_fused > 7) return fail(SNICIT_E_INVALID_ARG, "bad pre_fused");
    if (opt.pre_const < 0 || opt.pre_const > 2) return fail(SNICIT_E_INVALID_ARG, "bad pre_const");
    if (opt.res_sparse < 0 || opt.res_sparse > 1) return fail(SNICIT_E_INVALID_ARG, "bad res_sparse");
    if (opt.dyn_t < 0 || opt.dyn_t > 1) return fail(SNICIT_E_INVALID_ARG, "bad dyn_t");
    if (opt.kernel == SNICIT_KERNEL_ELL && !net->has_ell)
        return fail(SNICIT_E_UNSUPPORTED, "network loaded in compact circulant form has no ELL copy");
    const int N = net->N, L = net->L;
    if (opt.kernel == SNICIT_KERNEL_CIRC || opt.kernel == SNICIT_KERNEL_CIRC_SMEM)
        for (int l = 0; l < L; ++l)
            if (net->plan[l].kind == 0)
                return fail(SNICIT_E_UNSUPPORTED, "layer " + std::to_string(l) + " is not circulant");
    const int R = (int)batch;
    int tt = std::min(t, L);
    const int n_seg = opt.n_segments == 0 ? N : opt.n_segments;
    const int ne_interval = opt.ne_interval > 0 ? opt.ne_interval : 64;
    DeviceGuard dg(net->device);
    CUDA_TRY(dg.status);
    CUDA_TRY(ensure_workspace(net, R, s, n_seg));
    cudaStream_t st = net->stream;
    int64_t launches = y0_mode == 2 ? 1 : 0;  // + the unpack kernel of snicit_infer_packed (mode 2)
    int circ_layers = 0;
    net->have_result = false;
    net->ev_map = net->ev_res = false;
    net->dyn_pre = net->dyn_post = false;
    snicit_stats_t stats{};
    stats.batch = batch;
    stats.threshold_layer = tt;

    if (opt.timing) CUDA_TRY(cudaEventRecord(net->ev[0], st));
    bool host_streamed = false;  // host fp32 rows uploaded by stream_upload while the pre phase runs
    // ---- input
    const float* cur;
    float* bufs[2] = {net->Ya.p, net->Yb.p};
    int nxt_i = 0;
    if (y0_on_device) {
        cur = y0;
    } else if (y0_mode == 3) {
        cur = nullptr;  // the row-resident kernel reads the packed rows itself
    } else {
        if (y0_mode == 1 && R > 0) {
            int H_ = 0, g_ = 0;
            if (!opt.dyn_t && pf_plan(net, tt, opt, R, &H_, &g_)) {  // the row-resident kernel polls the chunks' flags
                CUDA_TRY(stream_upload(net, net->Ya.p, y0, sizeof(float) * (size_t)N, R, &bits_ready, &ready_rows));
                host_streamed = true;
            } else {
                CUDA_TRY(cudaMemcpyAsync(net->Ya.p, y0, sizeof(float) * (size_t)R * N, cudaMemcpyHostToDevice, st));
            }
        }
        cur = net->Ya.p;
        nxt_i = 1;
    }
    // ---- dynamic threshold layer (options.dyn_t): t is chosen from the first s rows before the pre phase
    if (opt.dyn_t && tt > 0 && R > 0) {
        int chosen = tt;
        CUDA_TRY(choose_t(net, cur, y0_mode == 3 ? bits : nullptr, one, R, s, tt, &chosen));
        tt = chosen;
        stats.threshold_layer = tt;
        launches += 2 * net->probe_layers + 2;
    }
    int* cnt = net->counters.p;
    int* scratch = net->cscratch.p;
    int* lists[2] = {net->list0.p, net->list1.p};
    int li = 0;                                         // lists[li] is the active-row list
    const int live_ctr[3] = {CNT_LIVE0, CNT_LIVE1, CNT_LIVE2};
    int ci = 0;                                         // cnt + live_ctr[ci] is its length
    CUDA_TRY(launch_iota(lists[0], R, cnt + CNT_LIVE0, st));
    CUDA_TRY(cudaMemsetAsync(cnt + CNT_LIVE1, 0, sizeof(int), st));
    launches += 1;
    const bool drop = opt.drop_dead_rows != 0;
    // zero input rows are dead only when the conversion happens at t = 0 (otherwise layer 0 drops them)
    if (drop && net->dead_ok[0] && tt == 0 && R > 0) {
        CUDA_TRY(launch_row_nonzero(cur, N, lists[li], cnt + live_ctr[ci], net->flag_pos.p, R, net->num_sms, st));
        CUDA_TRY(launch_compact(lists[li], cnt + live_ctr[ci], net->flag_pos.p, lists[li ^ 1],
                                cnt + live_ctr[(ci + 1) % 3], R, scratch, st));
        launches += 3;
        CUDA_TRY(cudaMemsetAsync(cnt + live_ctr[(ci + 2) % 3], 0, sizeof(int), st));
        li ^= 1;
        ci = (ci + 1) % 3;
    }
    // ---- a1: pre-convergence layers, Eq. 1 for i = 0..t-1
    const bool prof = opt.timing >= 2;
    if (prof) {
        while ((int)net->lev.size() < 2 * tt) {
            cudaEvent_t e;
            CUDA_TRY(cudaEventCreate(&e));
            net->lev.push_back(e);
        }
        CUDA_TRY(net->hist.ensure(std::max(tt, 1)));
        net->prof_layers = tt;
    } else {
        net->prof_layers = 0;
    }
    // row-resident fused pre phase (kernels_pre_fused.cu): one launch for layers 0..t-1
    int pf_H = 96, pf_gen = 0;
    bool pf_cluster = false, pf_bits_ok = true;
    const bool pf = pf_plan(net, tt, opt, R, &pf_H, &pf_gen, &pf_cluster, &pf_bits_ok);
    if (y0_mode == 3 && pf && !pf_bits_ok) return fail(SNICIT_E_STATE, "packed rows not readable by the pre-phase kernel");
    if (y0_mode == 3 && !pf && R > 0) return fail(SNICIT_E_STATE, "packed rows without the row-resident kernel");
    net->last_pre_fused = pf;
    const int dead_zeroed = (pf && y_out_on_device && y_out && drop) ? 1 : 0;  // y_out rows of dead rows
    // a device y_out holds Y(t) too (the row-resident kernel writes it there): rows whose Y(L) equals
    // their constant Y(t) are then never rewritten by the recovery (unless y0 overlaps y_out)
    const bool yt_out = pf && y_out_on_device && y_out &&
                        !(y0_on_device && y0 && (const char*)y0 < (const char*)(y_out + (size_t)R * N) &&
                          (const char*)y_out < (const char*)(y0 + (size_t)R * N));
    net->last_dead_zeroed = dead_zeroed != 0;
    stats.pre_fused = pf ? (pf_cluster ? 2 : 1) : 0;
    if (R > 0) CUDA_TRY(cudaMemsetAsync(net->rconst.p, 0, (size_t)R, st));  // rows constant at t (R26)
    if (pf) {
        if (prof) {
            CUDA_TRY(cudaMemcpyAsync(net->hist.p, cnt + live_ctr[ci], sizeof(int), cudaMemcpyDeviceToDevice, st));
            CUDA_TRY(cudaEventRecord(net->lev[0], st));
            net->prof_layers = 1;
        }
        CUDA_TRY(cudaMemsetAsync(cnt + CNT_PFWORK, 0, 2 * sizeof(int), st));
        CUDA_TRY(cudaMemsetAsync(net->pf_full.p, 0, 2 * sizeof(unsigned long long), st));
        PreFusedArgs pa{};
        pa.N = N;
        pa.t = tt;
        pa.H = pf_H;
        pa.ymax = net->ymax;
        pa.drop = drop ? 1 : 0;
        pa.const_skip = opt.pre_fused != 2 ? 1 : 0;
        pa.range_pred = opt.pre_fused != 6 ? 1 : 0;  // R30 / R31 (6: R26 alone, for measurement)
        {  // R34 with R30 / R31 (SNICIT_WINB=0: off, for A/B measurement)
            static const bool winb_off = [] {
                const char* e = getenv("SNICIT_WINB");
                return e && e[0] == '0';
            }();
            pa.win_bounds = pa.range_pred && !winb_off ? 1 : 0;
        }
        // R32: packed rows (1, 3, 5), every two-valued row (7), never (2, 6: fma chains only)
        // (1 also by default for fp32 rows at N = 2048..4096: several CTAs per SM hide the bitmap build and its
        // barriers -- C2 1.26 -> 1.15 ms; at N = 16384, one CTA per SM, it is slower: 3.91 -> 4.47 ms, and
        // at N = 1024 (C1, 2000 rows) 0.30 -> 0.33 ms)
        pa.popc0 = (opt.pre_fused == 6 || opt.pre_fused == 2) ? 0
                   : (opt.pre_fused == 7 || (opt.pre_fused == 1 && N >= 2048 && N <= 4096)) ? 1 : 2;
        pa.gen_str = pf_gen;
        pa.yin = cur;
        pa.ybits = y0_mode == 3 ? bits : nullptr;
        pa.one = one;
        pa.ready = (y0_mode == 3 || host_streamed) ? bits_ready : nullptr;
        pa.ready_rows = ready_rows;
        pa.yout = yt_out ? y_out : bufs[nxt_i];
        pa.rows = lists[li];
        pa.count = cnt + live_ctr[ci];
        pa.app_list = drop ? lists[li ^ 1] : nullptr;
        pa.app_count = cnt + live_ctr[(ci + 1) % 3];
        pa.work = cnt + CNT_PFWORK;
        pa.full_rl = net->pf_full.p;
        pa.ydead = (y_out_on_device && y_out && drop) ? y_out : nullptr;
        pa.rconst = net->rconst.p;
        pa.rval = net->rval.p;
        pa.n_const = cnt + CNT_PFCONST;
        if (opt.timing) {
            CUDA_TRY(net->dynbuf.ensure((size_t)2 * (tt + 1) + 2 * (L + 1)));
            CUDA_TRY(cudaMemsetAsync(net->dynbuf.p, 0, sizeof(unsigned long long) * 2 * (tt + 1), st));
            pa.dyn = net->dynbuf.p;
            net->dyn_pre = true;
        }
        if (pf_cluster)
            CUDA_TRY(launch_pre_cluster(pa, net->pf_layers_h.data(), net->num_sms, st));
        else if (opt.pre_fused == 5)
            CUDA_TRY(launch_pre_pair(pa, net->pf_layers_h.data(), net->num_sms, st));
        else
            CUDA_TRY(launch_pre_fused(pa, net->pf_layers_h.data(), net->num_sms, st));
        if (host_streamed) CUDA_TRY(cudaStreamWaitEvent(st, net->cev[1], 0));  // Ya reused after this
        if (prof) CUDA_TRY(cudaEventRecord(net->lev[1], st));
        ++launches;
        circ_layers += tt;
        net->last_kernel_circ = true;
        if (yt_out) {
            cur = y_out;  // both workspace buffers stay free for the residues
        } else {
            cur = bufs[nxt_i];
            nxt_i ^= 1;
        }
        if (drop) {
            li ^= 1;
            ci = (ci + 1) % 3;
        }
    }
    // constant-row mode of the per-layer path (R26, kernels_const.cu): every layer < t circulant with
    // uniform weight and bias and run by the column-streaming or segmented kernel
    bool pcst = !pf && opt.pre_const != 0 && tt > 0 && R > 0 && opt.kernel == SNICIT_KERNEL_AUTO;
    for (int l = 0; l < tt && pcst; ++l)
        pcst = (net->pf_elig[l] != 0 && (use_col(net, l, opt.kernel) || use_seg(net, l, opt.kernel))) ||
               ell_const_ok(net, l, opt.kernel);
    net->last_pre_const = pcst;
    if (pcst) CUDA_TRY(cudaMemsetAsync(cnt + CNT_CCOUNT, 0, sizeof(int), st));
    // range prediction (R30) in constant-row mode: horizon tables when layers 0..t-1 share weight and bias
    float thr_hi[kRangeK], thr_lo[kRangeK];
    const bool thr_ok = pcst && opt.pre_const != 2 && range_tables(net->pf_layers_h.data(), tt, net->ymax, thr_hi, thr_lo);
    for (int l = 0; l < tt && !pf; ++l) {
        // exact dead-row compaction (R23) fused into the layer: rows with a non-zero output are
        // appended (unordered) to the other list; the append counter of the NEXT dropping layer is
        // zeroed by this one (rotating counters), so no extra launch is needed.  Constant-row mode:
        // the list changes at every layer (constant rows leave it)
        const bool dead_now = drop && net->dead_ok[l + 1];
        const bool drop_now = dead_now || pcst;
        if (prof) {
            CUDA_TRY(cudaMemcpyAsync(net->hist.p + l, cnt + live_ctr[ci], sizeof(int), cudaMemcpyDeviceToDevice, st));
            CUDA_TRY(cudaEventRecord(net->lev[2 * l], st));
        }
        LayerArgs a = layer_args(net, l, opt.kernel == SNICIT_KERNEL_ELL);
        a.yin = cur;
        a.yout = bufs[nxt_i];
        a.rows = lists[li];
        a.count = cnt + live_ctr[ci];
        // segmented layers: row flags OR-ed across CTAs + a compaction launch; the others append
        // segmented layers (and general layers in constant-row mode): per-row flags / output ranges, then a
        // separate compaction or split launch instead of the fused append
        const bool seg = (use_seg(net, l, opt.kernel) && !use_col(net, l, opt.kernel)) ||
                         (pcst && !use_circ(net, l, opt.kernel));
        a.row_ctr = net->rowctr.p;                     // column-streaming kernel: last warp of a row appends
        if (drop_now && !seg) {
            a.app_list = lists[li ^ 1];
            a.app_count = cnt + live_ctr[(ci + 1) % 3];
            a.zero_count = cnt + live_ctr[(ci + 2) % 3];
        }
        if (drop_now && seg && !pcst) a.flag_pos = net->segflag.p;
        if (pcst) {
            a.cmin = net->cmin.p;
            a.cmax = net->cmax.p;
            a.clist = net->clist.p;
            a.cval = net->cval.p;
            a.clayer = net->clayer.p;
            a.ccount = cnt + CNT_CCOUNT;
            a.layer = l;
            a.dead_drop = dead_now ? 1 : 0;
            if (thr_ok && l + 1 < tt) {  // k = t - 1 - l layers follow this one
                const int k = std::min(tt - 1 - l, kRangeK);
                a.thr_hi = thr_hi[k - 1];
                a.thr_lo = thr_lo[k - 1];
                a.thr_layer = tt - 1;
                a.thr_dead = (drop && net->dead_ok[tt]) ? 1 : 0;
            }
        }
        CUDA_TRY(run_layer(net, l, opt.kernel, MODE_PLAIN, a, R));
        if (prof) CUDA_TRY(cudaEventRecord(net->lev[2 * l + 1], st));
        ++launches;
        if (pcst && seg) {
            CUDA_TRY(launch_const_split(lists[li], cnt + live_ctr[ci], net->cmin.p, net->cmax.p, lists[li ^ 1],
                                        cnt + live_ctr[(ci + 1) % 3], net->clist.p, net->cval.p, net->clayer.p,
                                        cnt + CNT_CCOUNT, l, dead_now ? 1 : 0, R, st, &a));
            CUDA_TRY(cudaMemsetAsync(cnt + live_ctr[(ci + 2) % 3], 0, sizeof(int), st));
            launches += 1;
        } else if (drop_now && seg) {
            CUDA_TRY(launch_compact(lists[li], cnt + live_ctr[ci], net->segflag.p, lists[li ^ 1],
                                    cnt + live_ctr[(ci + 1) % 3], R, scratch, st, 1));
            CUDA_TRY(cudaMemsetAsync(cnt + live_ctr[(ci + 2) % 3], 0, sizeof(int), st));
            launches += 2;
        }
        circ_layers += use_circ(net, l, opt.kernel);
        net->last_kernel_circ = use_circ(net, l, opt.kernel);
        cur = bufs[nxt_i];
        nxt_i ^= 1;
        if (drop_now) {
            li ^= 1;
            ci = (ci + 1) % 3;
        }
    }
    if (pcst) {  // constant rows through the remaining layers (scalar chains), written once, relisted
        CUDA_TRY(launch_const_finish(net->clist.p, net->cval.p, net->clayer.p, cnt + CNT_CCOUNT, net->pf_layers_d.p, tt,
                                     net->ymax, drop ? 1 : 0, N, bufs[nxt_i ^ 1], lists[li], cnt + live_ctr[ci],
                                     net->num_sms, st, net->rconst.p, net->rval.p));
        ++launches;
    }
    int* list_cur = lists[li];
    int* cnt_cur = cnt + live_ctr[ci];
    int* list_nxt = lists[li ^ 1];
    if (opt.timing) CUDA_TRY(cudaEventRecord(net->ev[1], st));
    // live flags at t (recovery of the plain path, ordered live list, debug hook)
    CUDA_TRY(launch_fill_u8(net->live_row.p, R, 0, st));
    CUDA_TRY(launch_mark_rows(list_cur, cnt_cur, net->live_row.p, R, st));
    CUDA_TRY(launch_fill_i32(cnt + CNT_ALL, 1, R, st));
    launches += 3;

    float* y_dst = y_out_on_device ? y_out : nullptr;
    const float* yfinal = cur;
    const float* cfinal = net->cbuf0.p;
    const bool converted = tt < L;
    net->last_converted = converted;
    net->last_const = false;
    if (!converted) {
        if (opt.timing) {
            CUDA_TRY(cudaEventRecord(net->ev[2], st));
            CUDA_TRY(cudaEventRecord(net->ev[3], st));
        }
        if (!y_out_on_device && y_out) y_dst = bufs[nxt_i];
        CUDA_TRY(launch_recover(N, R, 1, yfinal, net->live_row.p, nullptr, nullptr, nullptr, nullptr, y_dst,
                                net->cat.p, net->num_sms, st, y_dst == y_out ? dead_zeroed : 0,
                                yt_out ? net->rconst.p : nullptr, net->rval.p, nullptr));
        ++launches;
    } else {
        // ordered live list: "the first s columns" are the first s live rows by id (R14)
        CUDA_TRY(launch_compact(nullptr, cnt + CNT_ALL, net->live_row.p, list_nxt, cnt + CNT_ORD, R, scratch, st));
        launches += 2;
        list_cur = list_nxt;
        cnt_cur = cnt + CNT_ORD;
        // ---- a2/a3: sampling + sum downsampling + Alg. 1 pruning -> y*
        CUDA_TRY(launch_downsample(cur, N, list_cur, cnt_cur, s, n_seg, net->F.p, st));
        // (Alg. 1's pair counts go to the Alg. 2 distance buffer: rows x s ints >= s_eff x s, unused until a4)
        CUDA_TRY(launch_prune(net->F.p, cnt_cur, s, n_seg, opt.eta, opt.eps, list_cur, net->cent.p, cnt + CNT_NCENT,
                              cnt + CNT_SEFF, net->col_idx.p, net->dist.p, st));
        // ---- a4: mapper + residues (Alg. 2); dead rows keep M = -2
        CUDA_TRY(launch_fill_i32(net->M.p, R, -2, st));
        CUDA_TRY(launch_fill_u8(net->ne_row.p, R, 0, st));
        float* yhat = bufs[nxt_i];
        float* yhat_other = bufs[nxt_i ^ 1];
        CUDA_TRY(cudaMemsetAsync(net->ctr64.p, 0, sizeof(unsigned long long) * C64_N, st));
        if (opt.timing) CUDA_TRY(cudaEventRecord(net->ev[6], st));
        CUDA_TRY(launch_map_residual(cur, N, list_cur, cnt_cur, net->cent.p, cnt + CNT_NCENT, net->M.p, net->cslot.p,
                                     net->ne_row.p, net->flag_pos.p, yhat, net->cbuf0.p, R, net->num_sms, st,
                                     net->rconst.p, net->rval.p, net->ctr64.p + C64_RES_NNZ, net->dist.p, s,
                                     net->rnnz.p, net->need.p, cnt + CNT_NEED));
        if (opt.timing) CUDA_TRY(cudaEventRecord(net->ev[7], st));
        net->ev_map = opt.timing != 0;
        int* rlist = net->res0.p;
        int* rlist_nxt = net->res1.p;
        int* rcnt = cnt + CNT_RES0;
        int* rcnt_nxt = cnt + CNT_RES1;
        CUDA_TRY(launch_compact(list_cur, cnt_cur, net->flag_pos.p, rlist, rcnt, R, scratch, st));
        CUDA_TRY(launch_iota(net->iota_s.p, s, nullptr, st));
        CUDA_TRY(cudaMemcpyAsync(net->ne_t.p, net->ne_row.p, (size_t)R, cudaMemcpyDeviceToDevice, st));
        launches += 7;
        if (opt.timing) CUDA_TRY(cudaEventRecord(net->ev[2], st));
        // ---- a5: post-convergence layers, Eq. 5 for i = t..L-1
        float* c_cur = net->cbuf0.p;
        float* c_nxt = net->cbuf1.p;
        float* yh_cur = yhat;
        float* yh_nxt = yhat_other;
        // general (non-circulant) post layers with a general-CSC kernel schedule run per layer: the tiled
        // kernel (kernels_gen.cu) beats the fused trajectory kernels' per-row gathers on them
        bool gen_post = false;
        for (int l = tt; l < L; ++l) gen_post |= !use_circ(net, l, opt.kernel) && net->plan[l].gen && net->grl > 0;
        const bool fused = opt.post_mode == 0 && N <= post_fused_max_n() && !(gen_post && gen_enabled());
        // fused mode: no host read of the residue count (the kernels read it on the device and the
        // a_c rows are written only when residue rows exist), so the stream is never stalled here;
        // res_host = 1 means "maybe"
        int res_host = 1;
        if (!fused) CUDA_TRY(read_counter(net, CNT_RES0, &res_host));
        if (!fused) stats.residual_at_t = res_host;
        net->res_at_t_lazy = fused;  // fused: CNT_RES0 still holds it when snicit_stats reads it
        net->last_fused = fused;
        // constant centroid rows (centroid_const_kernel): every post layer circulant with uniform
        // weights and bias.  Fused mode: in place, the trajectory kernels skip the carried rows.
        // Per-layer mode (no residues): into cbuf1; the layer loop is skipped when all were carried.
        bool const_ok = opt.post_const != 0 && opt.kernel != SNICIT_KERNEL_ELL;
        // (any layer whose columns all hold K = 32 entries of one weight, with one bias: every output of a
        // constant row evaluates the same stored-order chain -- circulant or not, R25)
        for (int l = tt; l < L && const_ok; ++l)
            const_ok = net->plan[l].uniform && net->plan[l].ubias && !net->plan[l].ragged && net->plan[l].K == 32;
        int* cdone = nullptr;
        bool all_const = false;
        if (const_ok && (fused || res_host == 0)) {
            CUDA_TRY(net->cdone.ensure((size_t)s));
            cdone = net->cdone.p;
            CUDA_TRY(cudaMemsetAsync(cnt + CNT_CDONE, 0, sizeof(int), st));
            PostArgs pc{};
            pc.N = N;
            pc.L = L;
            pc.t = tt;
            pc.ymax = net->ymax;
            pc.layers = net->post_layers_d.p;
            pc.cbuf = net->cbuf0.p;
            pc.n_cent = cnt + CNT_NCENT;
            pc.s = s;
            if (fused && res_host > 0) {
                CUDA_TRY(net->a_all.ensure((size_t)(L - tt) * (size_t)s * N));
                pc.a_all = net->a_all.p;
                pc.rcount = rcnt;
            }
            CUDA_TRY(launch_centroid_const(pc, fused ? net->cbuf0.p : net->cbuf1.p, cdone, cnt + CNT_CDONE, s, st));
            ++launches;
            if (!fused) {
                int nd = 0, nc = 0;
                CUDA_TRY(read_counter(net, CNT_CDONE, &nd));
                CUDA_TRY(read_counter(net, CNT_NCENT, &nc));
                all_const = nd == nc;
                if (all_const) {
                    c_cur = net->cbuf1.p;
                    c_nxt = net->cbuf0.p;
                    for (int l = tt; l < L; ++l) circ_layers += use_circ(net, l, opt.kernel);
                }
            }
        }
        net->last_const = cdone != nullptr;
        if (fused) {
            // centroid trajectories (+ a_c per layer when residue rows exist), then residue rows
            PostArgs pa{};
            pa.N = N;
            pa.L = L;
            pa.t = tt;
            pa.ymax = net->ymax;
            pa.prune_eps = opt.prune_eps;
            pa.layers = net->post_layers_d.p;
            pa.cbuf = net->cbuf0.p;
            pa.n_cent = cnt + CNT_NCENT;
            pa.s = s;
            if (res_host > 0) {
                CUDA_TRY(net->a_all.ensure((size_t)(L - tt) * (size_t)s * N));
                pa.a_all = net->a_all.p;
            }
            pa.rlist = rlist;
            pa.rcount = rcnt;
            pa.work_counter = cnt + CNT_WORK;
            pa.yhat = yhat;
            pa.cslot = net->cslot.p;
            pa.ne_row = net->ne_row.p;
            pa.alive_count = cnt + CNT_ALIVE;
            pa.cdone = cdone;
            pa.ctr64 = net->ctr64.p;
            pa.res_sparse = opt.res_sparse;
            pa.rnnz = net->rnnz.p;
            if (opt.timing) {
                CUDA_TRY(net->dynbuf.ensure((size_t)2 * (tt + 1) + 2 * (L + 1)));
                unsigned long long* d = net->dynbuf.p + 2 * (tt + 1);
                CUDA_TRY(cudaMemsetAsync(d, 0, sizeof(unsigned long long) * 2 * (L - tt + 1), st));
                pa.dyn = d;
                net->dyn_post = true;
            }
            CUDA_TRY(cudaMemsetAsync(cnt + CNT_WORK, 0, 2 * sizeof(int), st));
            pa.force_ell = opt.kernel == SNICIT_KERNEL_ELL ? 1 : 0;
            // cluster (DSMEM) trajectory when every post layer is circulant and partition-compatible
            std::vector<int> nus(L, 0), clss(L, -1);
            int win_max = 0;
            for (int l = 0; l < L; ++l) {
                if (use_circ(net, l, opt.kernel)) {
                    nus[l] = net->plan[l].nu;
                    clss[l] = circ_class_of(N, nus[l]);
                    const int S8 = N / 8;
                    const int w = clss[l] == 0 ? S8 + 40 : (clss[l] == 1 ? S8 : (S8 / nus[l] + 32) * nus[l]);
                    if (l >= tt) win_max = std::max(win_max, w);
                }
            }
            const bool use_cluster = opt.post_cluster != 0 && centroid_cluster_ok(N, nus.data(), clss.data(), tt, L);
            {  // every post layer circulant with one weight and one bias: constant rows stay constant (R25)
                bool sok = opt.post_const != 0 && opt.kernel == SNICIT_KERNEL_AUTO;
                for (int l = tt; l < L && sok; ++l) sok = net->pf_elig[l] != 0;
                pa.scalar_ok = sok ? 1 : 0;
            }
            net->last_cluster = use_cluster;
            if (use_cluster)
                CUDA_TRY(launch_centroid_cluster(pa, s, win_max, st));
            else
                CUDA_TRY(launch_centroid_traj(pa, s, st));
            ++launches;
            for (int l = tt; l < L; ++l) circ_layers += use_circ(net, l, opt.kernel);
            if (res_host > 0) {
                bool sok = opt.post_const != 0 && opt.kernel == SNICIT_KERNEL_AUTO;
                for (int l = tt; l < L && sok; ++l) sok = net->pf_elig[l] != 0;
                if (sok) {  // constant residue rows over constant centroids leave as scalars
                    CUDA_TRY(net->cfrom.ensure((size_t)s));
                    CUDA_TRY(net->acs.ensure((size_t)s * (L - tt)));
                    pa.cfrom = net->cfrom.p;
                    pa.acs = net->acs.p;
                    pa.wb = net->wb_d.p;
                    pa.scalar_ok = 1;
                    CUDA_TRY(launch_acconst(pa, s, st));
                    ++launches;
                }
                if (opt.timing) CUDA_TRY(cudaEventRecord(net->ev[8], st));
                CUDA_TRY(launch_residual_traj(pa, R, net->num_sms, st));
                if (opt.timing) CUDA_TRY(cudaEventRecord(net->ev[9], st));
                net->ev_res = opt.timing != 0;
                ++launches;
            }
        }
        for (int l = tt; l < L && !fused && !all_const; ++l) {
            // centroids: Eq. 5 first case, keep a_c
            LayerArgs a = layer_args(net, l, opt.kernel == SNICIT_KERNEL_ELL);
            a.yin = c_cur;
            a.yout = c_nxt;
            a.rows = net->iota_s.p;
            a.count = cnt + CNT_NCENT;
            a.a_out = net->ac.p;
            CUDA_TRY(run_layer(net, l, opt.kernel, MODE_CENTROID, a, s));
            ++launches;
            circ_layers += use_circ(net, l, opt.kernel);
            if (res_host > 0) {
                // residues: Eq. 5 second case, only non-empty rows (ne_idx)
                LayerArgs b = layer_args(net, l, opt.kernel == SNICIT_KERNEL_ELL);
                b.yin = yh_cur;
                b.yout = yh_nxt;
                b.rows = rlist;
                b.count = rcnt;
                b.a_c = net->ac.p;
                b.cslot = net->cslot.p;
                b.prune_eps = opt.prune_eps;
                if (use_seg(net, l, opt.kernel)) {  // flags OR-ed across segments; ne_rec set by the compaction
                    b.flag_pos = net->segflag.p;
                    CUDA_TRY(run_layer(net, l, opt.kernel, MODE_RESIDUAL, b, R));
                    CUDA_TRY(launch_compact(rlist, rcnt, net->segflag.p, rlist_nxt, rcnt_nxt, R, scratch, st, 1,
                                            net->ne_row.p));
                } else {
                    b.flag_pos = net->flag_pos.p;
                    b.flag_row = net->ne_row.p;
                    CUDA_TRY(run_layer(net, l, opt.kernel, MODE_RESIDUAL, b, R));
                    CUDA_TRY(launch_compact(rlist, rcnt, net->flag_pos.p, rlist_nxt, rcnt_nxt, R, scratch, st));
                }
                launches += 2;
                std::swap(rlist, rlist_nxt);
                std::swap(rcnt, rcnt_nxt);
                std::swap(yh_cur, yh_nxt);
                if (((l - tt + 1) % ne_interval) == 0) {
                    const int which = (rcnt == cnt + CNT_RES0) ? CNT_RES0 : CNT_RES1;
                    CUDA_TRY(read_counter(net, which, &res_host));
                }
            }
            std::swap(c_cur, c_nxt);
        }
        if (opt.timing) CUDA_TRY(cudaEventRecord(net->ev[3], st));
        net->res_final_counter = -1;
        if (res_host > 0) net->res_final_counter = fused ? CNT_ALIVE : ((rcnt == cnt + CNT_RES0) ? CNT_RES0 : CNT_RES1);
        stats.residual_final = 0;
        yfinal = yh_cur;
        cfinal = c_cur;
        // ---- a6: recovery (Eq. 6)
        if (!y_out_on_device && y_out) y_dst = yh_nxt;  // free buffer
        CUDA_TRY(launch_recover(N, R, 0, yfinal, nullptr, net->M.p, net->cslot.p, net->ne_row.p, cfinal, y_dst,
                                net->cat.p, net->num_sms, st, y_dst == y_out ? dead_zeroed : 0,
                                (yt_out && y_dst == y_out) ? net->rconst.p : nullptr, net->rval.p, cdone));
        ++launches;
    }
    // categories: ordered compaction of the cat flags over all rows (R13)
    CUDA_TRY(launch_compact(nullptr, cnt + CNT_ALL, net->cat.p, net->catlist.p, cnt + CNT_NCAT, R, scratch, st));
    launches += 2;
    if (opt.timing) CUDA_TRY(cudaEventRecord(net->ev[4], st));
    if (!y_out_on_device && y_out && R > 0)
        CUDA_TRY(cudaMemcpyAsync(y_out, y_dst, sizeof(float) * (size_t)R * N, cudaMemcpyDeviceToHost, st));
    if (opt.timing) CUDA_TRY(cudaEventRecord(net->ev[5], st));
    net->have_result = true;
    net->last_batch = batch;
    net->last_offset = row_offset;
    net->last_t = tt;
    net->last_s = s;
    net->last_n = n_seg;
    stats.kernel_launches = launches;
    stats.circ_layers = circ_layers;
    net->stats = stats;
    if (!opt.timing) {
        net->stats.t_pre_ms = net->stats.t_convert_ms = net->stats.t_post_ms = net->stats.t_recover_ms = -1.0;
        net->stats.t_total_ms = -1.0;
    }
    net->live_counter = live_ctr[ci];
    if (opt.timing) {
        CUDA_TRY(cudaEventSynchronize(net->ev[5]));
        float ms;
        cudaEventElapsedTime(&ms, net->ev[0], net->ev[1]);
        net->stats.t_pre_ms = ms;
        cudaEventElapsedTime(&ms, net->ev[1], net->ev[2]);
        net->stats.t_convert_ms = ms;
        cudaEventElapsedTime(&ms, net->ev[2], net->ev[3]);
        net->stats.t_post_ms = ms;
        cudaEventElapsedTime(&ms, net->ev[3], net->ev[4]);
        net->stats.t_recover_ms = ms;
        cudaEventElapsedTime(&ms, net->ev[0], net->ev[5]);
        net->stats.t_total_ms = ms;
    }
    net->stats.t_map_ms = net->stats.t_residual_ms = -1.0;
    if (net->ev_map) {
        float ms;
        cudaEventElapsedTime(&ms, net->ev[6], net->ev[7]);
        net->stats.t_map_ms = ms;
    }
    if (net->ev_res) {
        float ms;
        cudaEventElapsedTime(&ms, net->ev[8], net->ev[9]);
        net->stats.t_residual_ms = ms;
    }
    // a host buffer is involved (y0 read by an async H2D copy, y_out filled by an async D2H copy):
    // return only when the caller may read / reuse it
    if (y0_mode == 1 || (y_out && !y_out_on_device)) CUDA_TRY(cudaStreamSynchronize(st));
    return SNICIT_OK;
}

snicit_status snicit_infer(snicit_network* net, const float* y0, int64_t batch, int32_t y0_on_device,
                           int64_t row_offset, int32_t t, int32_t s, const snicit_options* opt, float* y_out,
                           int32_t y_out_on_device) {
    return infer_core(net, y0, batch, y0_on_device ? 0 : 1, row_offset, t, s, opt, y_out, y_out_on_device);
}

snicit_status snicit_infer_packed(snicit_network* net, const uint32_t* y0_bits, int64_t batch, int32_t bits_on_device,
                                  float one_value, int64_t row_offset, int32_t t, int32_t s,
                                  const snicit_options* opt, float* y_out, int32_t y_out_on_device) {
    if (!net) return fail(SNICIT_E_INVALID_ARG, "net NULL");
    if (batch < 0 || batch > 0x7fffffffLL) return fail(SNICIT_E_INVALID_ARG, "batch out of range");
    if (batch > 0 && !y0_bits) return fail(SNICIT_E_INVALID_ARG, "y0_bits NULL");
    if (!std::isfinite(one_value)) return fail(SNICIT_E_INVALID_ARG, "one_value not finite");
    if (t < 0 || s < 1) return fail(SNICIT_E_INVALID_ARG, "threshold_layer < 0 or centroid_count < 1");
    if (bits_on_device && misaligned16(y0_bits)) return fail(SNICIT_E_INVALID_ARG, "device y0_bits must be 16-byte aligned");
    const int N = net->N;
    const int R = (int)batch;
    const size_t W = ((size_t)N + 31) / 32;
    DeviceGuard dg(net->device);
    CUDA_TRY(dg.status);
    const int n_seg = (opt && opt->n_segments > 0 && opt->n_segments <= N) ? opt->n_segments : N;
    CUDA_TRY(ensure_workspace(net, R, s, n_seg));
    const uint32_t* bits = y0_bits;
    snicit_options o;
    if (opt)
        o = *opt;
    else
        snicit_default_options(&o);
    int H = 0, gen = 0;
    bool cl = false, bits_ok = true;
    const bool direct = N % 128 == 0 && !o.dyn_t && pf_plan(net, std::min(t, net->L), o, R, &H, &gen, &cl, &bits_ok) &&
                        bits_ok;
    const int* ready = nullptr;
    int ready_rows = 0;
    bool streamed = false;
    if (!bits_on_device && R > 0) {
        CUDA_TRY(net->bits.ensure((size_t)R * W));
        if (direct) {
            // streamed upload (the copy engine delivers chunks while the row-resident kernel runs)
            CUDA_TRY(stream_upload(net, net->bits.p, y0_bits, sizeof(uint32_t) * W, R, &ready, &ready_rows));
            streamed = true;
        } else {
            CUDA_TRY(cudaMemcpyAsync(net->bits.p, y0_bits, sizeof(uint32_t) * (size_t)R * W, cudaMemcpyHostToDevice,
                                     net->stream));
        }
        bits = net->bits.p;
    }
    snicit_status stt;
    if (direct) {
        // the row-resident kernel expands each row's bits in shared memory (no fp32 Y0 in HBM)
        stt = infer_core(net, nullptr, batch, 3, row_offset, t, s, opt, y_out, y_out_on_device, bits, one_value, ready,
                         ready_rows);
    } else {
        if (R > 0) CUDA_TRY(launch_unpack_bits(bits, R, N, one_value, net->Ya.p, net->num_sms, net->stream));
        stt = infer_core(net, nullptr, batch, 2, row_offset, t, s, opt, y_out, y_out_on_device);
    }
    // later work on the handle's stream (and the next upload) is ordered after this upload
    if (streamed) CUDA_TRY(cudaStreamWaitEvent(net->stream, net->cev[1], 0));
    // host bits are read by asynchronous copies: return once they are consumed
    if (stt == SNICIT_OK && !bits_on_device && R > 0) CUDA_TRY(cudaStreamSynchronize(net->stream));
    return stt;
}

snicit_status snicit_categories(snicit_network* net, int64_t* rows, int64_t* count, int32_t rows_on_device) {
    if (!net || !count) return fail(SNICIT_E_INVALID_ARG, "net/count NULL");
    if (!net->have_result) return fail(SNICIT_E_STATE, "no inference result");
    DeviceGuard dg(net->device);
    CUDA_TRY(dg.status);
    int total = 0;
    CUDA_TRY(read_counter(net, CNT_NCAT, &total));
    if (!rows) {
        *count = total;
        return SNICIT_OK;
    }
    const int64_t n = std::min<int64_t>(*count, total);
    if (n > 0) {
        std::vector<int32_t> tmp((size_t)n);
        CUDA_TRY(cudaMemcpyAsync(tmp.data(), net->catlist.p, sizeof(int32_t) * n, cudaMemcpyDeviceToHost, net->stream));
        CUDA_TRY(cudaStreamSynchronize(net->stream));
        std::vector<int64_t> out((size_t)n);
        for (int64_t i = 0; i < n; ++i) out[i] = net->last_offset + tmp[i];
        if (rows_on_device)
            CUDA_TRY(cudaMemcpy(rows, out.data(), sizeof(int64_t) * n, cudaMemcpyHostToDevice));
        else
            memcpy(rows, out.data(), sizeof(int64_t) * n);
    }
    *count = n;
    return SNICIT_OK;
}

snicit_status snicit_categories_device(snicit_network* net, int64_t* out, int64_t capacity) {
    if (!net || !out) return fail(SNICIT_E_INVALID_ARG, "net/out NULL");
    if (capacity < 0) return fail(SNICIT_E_INVALID_ARG, "capacity < 0");
    if (reinterpret_cast<uintptr_t>(out) & 7u) return fail(SNICIT_E_INVALID_ARG, "out must be 8-byte aligned");
    if (!net->have_result) return fail(SNICIT_E_STATE, "no inference result");
    DeviceGuard dg(net->device);
    CUDA_TRY(dg.status);
    CUDA_TRY(launch_export_categories(net->catlist.p, net->counters.p + CNT_NCAT, (long long)net->last_offset,
                                      reinterpret_cast<long long*>(out), (long long)capacity, net->stream));
    return SNICIT_OK;
}

snicit_status snicit_stats(snicit_network* net, snicit_stats_t* out) {
    if (!net || !out) return fail(SNICIT_E_INVALID_ARG, "net/out NULL");
    if (!net->have_result) return fail(SNICIT_E_STATE, "no inference result");
    DeviceGuard dg(net->device);
    CUDA_TRY(dg.status);
    int v = 0;
    CUDA_TRY(read_counter(net, net->live_counter, &v));
    net->stats.live_at_t = v;
    CUDA_TRY(read_counter(net, CNT_NCAT, &v));
    net->stats.n_categories = v;
    if (net->last_converted && net->res_final_counter >= 0) {
        CUDA_TRY(read_counter(net, net->res_final_counter, &v));
        net->stats.residual_final = v;
    }
    if (net->last_converted && net->res_at_t_lazy) {
        CUDA_TRY(read_counter(net, CNT_RES0, &v));
        net->stats.residual_at_t = v;
    }
    if (net->last_converted) {
        CUDA_TRY(read_counter(net, CNT_NCENT, &v));
        net->stats.n_centroids = v;
        CUDA_TRY(read_counter(net, CNT_SEFF, &v));
        net->stats.n_sampled = v;
    }
    net->stats.const_centroids = 0;
    if (net->last_converted && net->last_const) {
        CUDA_TRY(read_counter(net, CNT_CDONE, &v));
        net->stats.const_centroids = v;
    }
    net->stats.pre_const_rows = 0;
    net->stats.pre_full_rows = 0;
    net->stats.pre_popc_rows = 0;
    if (net->last_pre_const) {
        CUDA_TRY(read_counter(net, CNT_CCOUNT, &v));
        net->stats.pre_const_rows = v;
    }
    net->stats.res_nnz_at_t = net->stats.res_full_rl = net->stats.res_sparse_rl = 0;
    net->stats.res_sparse_out = net->stats.res_scalar_rl = net->stats.map_rows = 0;
    if (net->last_converted) {
        unsigned long long c64[C64_N];
        CUDA_TRY(cudaMemcpyAsync(c64, net->ctr64.p, sizeof(c64), cudaMemcpyDeviceToHost, net->stream));
        CUDA_TRY(cudaStreamSynchronize(net->stream));
        net->stats.res_nnz_at_t = (int64_t)c64[C64_RES_NNZ];
        net->stats.res_full_rl = (int64_t)c64[C64_FULL_RL];
        net->stats.res_sparse_rl = (int64_t)c64[C64_SPARSE_RL];
        net->stats.res_sparse_out = (int64_t)c64[C64_SPARSE_OUT];
        net->stats.res_scalar_rl = (int64_t)c64[C64_SCALAR_RL];
        net->stats.map_rows = (int64_t)c64[C64_MAP_ROWS];
    }
    if (net->last_pre_fused) {
        CUDA_TRY(read_counter(net, CNT_PFCONST, &v));
        net->stats.pre_const_rows = v;
        unsigned long long f[2] = {0, 0};
        CUDA_TRY(cudaMemcpy(f, net->pf_full.p, sizeof(f), cudaMemcpyDeviceToHost));
        net->stats.pre_full_rows = (int64_t)f[0];
        net->stats.pre_popc_rows = (int64_t)f[1];
    }
    *out = net->stats;
    return SNICIT_OK;
}

snicit_status snicit_layer_profile(snicit_network* net, int32_t max, double* ms, int64_t* rows, double* bytes,
                                   int32_t* n) {
    if (!net) return fail(SNICIT_E_INVALID_ARG, "net NULL");
    if (!net->have_result) return fail(SNICIT_E_STATE, "no inference result");
    DeviceGuard dg(net->device);
    CUDA_TRY(dg.status);
    CUDA_TRY(cudaStreamSynchronize(net->stream));
    const int cnt = std::min<int>(std::max(max, 0), net->prof_layers);
    std::vector<int> h((size_t)std::max(cnt, 1));
    if (cnt > 0) CUDA_TRY(cudaMemcpy(h.data(), net->hist.p, sizeof(int) * cnt, cudaMemcpyDeviceToHost));
    for (int l = 0; l < cnt; ++l) {
        float t = 0.f;
        CUDA_TRY(cudaEventElapsedTime(&t, net->lev[2 * l], net->lev[2 * l + 1]));
        if (ms) ms[l] = t;
        if (rows) rows[l] = h[l];
        if (bytes && net->last_pre_fused) {
            // row-resident kernel: every input row read once, every row alive at t written once
            int live = 0;
            CUDA_TRY(read_counter(net, net->live_counter, &live));
            // (+ the zeros of the rows found dead, written into y_out when it is on the device)
            const double dead = net->last_dead_zeroed ? (double)h[l] - live : 0.0;
            bytes[l] = 4.0 * net->N * ((double)h[l] + live + dead) + sizeof(PreFusedLayer) * (double)net->last_t;
        } else if (bytes) {
            const LayerPlan& pl = net->plan[l];
            // algorithmic bytes: rows read + written, weights, bias
            double wb;
            if (pl.kind != 0 && net->last_kernel_circ)
                wb = 4.0 * pl.K;
            else
                wb = (double)pl.K * net->N * ((net->idx16 ? 2.0 : 4.0) + (pl.uniform ? 0.0 : 4.0));
            bytes[l] = 8.0 * (double)h[l] * net->N + wb + 4.0 * net->N;
        }
    }
    if (n) *n = cnt;
    return SNICIT_OK;
}

snicit_status snicit_dynamics(snicit_network* net, int32_t max, int64_t* pre_full, int64_t* pre_live,
                              int64_t* res_alive, int64_t* res_scalar, int32_t* n) {
    if (!net) return fail(SNICIT_E_INVALID_ARG, "net NULL");
    if (!net->have_result) return fail(SNICIT_E_STATE, "no inference result");
    DeviceGuard dg(net->device);
    CUDA_TRY(dg.status);
    const int L = net->L, t = net->last_t;
    const int cnt = std::min<int>(std::max(max, 0), L);
    std::vector<unsigned long long> h(net->dynbuf.n ? net->dynbuf.n : 1, 0ull);
    if (net->dyn_pre || net->dyn_post) {
        CUDA_TRY(cudaMemcpyAsync(h.data(), net->dynbuf.p, sizeof(unsigned long long) * net->dynbuf.n,
                                 cudaMemcpyDeviceToHost, net->stream));
        CUDA_TRY(cudaStreamSynchronize(net->stream));
    }
    std::vector<int> hist;
    if (!net->last_pre_fused && net->prof_layers > 0) {  // per-layer pre path with timing == 2: active rows
        hist.resize((size_t)net->prof_layers);
        CUDA_TRY(cudaMemcpy(hist.data(), net->hist.p, sizeof(int) * hist.size(), cudaMemcpyDeviceToHost));
    }
    const unsigned long long* F = h.data();               // rows by full-evaluation count [t + 1]
    const unsigned long long* E = h.data() + (t + 1);     // rows by end layer [t + 1]
    const int nl = L - t;
    const unsigned long long* A = h.data() + 2 * (t + 1);          // residue rows by layers survived [nl + 1]
    const unsigned long long* Sc = A + (nl + 1);                    // residue rows by scalar start [nl + 1]
    for (int l = 0; l < cnt; ++l) {
        int64_t pf = -1, pl = -1, ra = -1, rs = -1;
        if (l < t && net->dyn_pre) {
            pf = pl = 0;
            for (int f = l + 1; f <= t; ++f) pf += (int64_t)F[f];
            for (int e = l + 1; e <= t; ++e) pl += (int64_t)E[e];
        } else if (l < t && l < (int)hist.size()) {
            pf = hist[l];
            if (l + 1 < (int)hist.size()) pl = hist[l + 1];
        }
        if (l >= t && net->dyn_post) {
            const int k = l - t;
            ra = rs = 0;
            for (int e = k + 1; e <= nl; ++e) ra += (int64_t)A[e];
            for (int c = 0; c <= k; ++c) rs += (int64_t)Sc[c];
        }
        if (pre_full) pre_full[l] = pf;
        if (pre_live) pre_live[l] = pl;
        if (res_alive) res_alive[l] = ra;
        if (res_scalar) res_scalar[l] = rs;
    }
    if (n) *n = cnt;
    return SNICIT_OK;
}

snicit_status snicit_debug_clustering(snicit_network* net, int32_t* cent, int32_t* n_cent, int32_t* M, uint8_t* ne_t,
                                      double* F, int32_t* n_sampled, uint8_t* live_t) {
    if (!net) return fail(SNICIT_E_INVALID_ARG, "net NULL");
    if (!net->have_result) return fail(SNICIT_E_STATE, "no inference result");
    DeviceGuard dg(net->device);
    CUDA_TRY(dg.status);
    CUDA_TRY(cudaStreamSynchronize(net->stream));
    const int R = (int)net->last_batch;
    int C = 0, se = 0;
    if (net->last_converted) {
        CUDA_TRY(cudaMemcpy(&C, net->counters.p + CNT_NCENT, sizeof(int), cudaMemcpyDeviceToHost));
        CUDA_TRY(cudaMemcpy(&se, net->counters.p + CNT_SEFF, sizeof(int), cudaMemcpyDeviceToHost));
    }
    if (n_cent) *n_cent = C;
    if (n_sampled) *n_sampled = se;
    if (cent && C > 0) CUDA_TRY(cudaMemcpy(cent, net->cent.p, sizeof(int) * C, cudaMemcpyDeviceToHost));
    if (M && R > 0 && net->last_converted) CUDA_TRY(cudaMemcpy(M, net->M.p, sizeof(int) * R, cudaMemcpyDeviceToHost));
    if (ne_t && R > 0 && net->last_converted) CUDA_TRY(cudaMemcpy(ne_t, net->ne_t.p, R, cudaMemcpyDeviceToHost));
    if (live_t && R > 0) CUDA_TRY(cudaMemcpy(live_t, net->live_row.p, R, cudaMemcpyDeviceToHost));
    if (F && se > 0) {
        std::vector<double> tmp((size_t)net->last_n * net->last_s);
        CUDA_TRY(cudaMemcpy(tmp.data(), net->F.p, sizeof(double) * tmp.size(), cudaMemcpyDeviceToHost));
        for (int g = 0; g < net->last_n; ++g)
            for (int q = 0; q < se; ++q) F[(size_t)g * se + q] = tmp[(size_t)g * net->last_s + q];
    }
    return SNICIT_OK;
}

snicit_status snicit_debug_layer(snicit_network* net, int32_t layer, const float* yin, float* yout, int64_t rows,
                                 int32_t kernel) {
    if (!net || !yin || !yout) return fail(SNICIT_E_INVALID_ARG, "NULL argument");
    if (layer < 0 || layer >= net->L) return fail(SNICIT_E_INVALID_ARG, "bad layer");
    if (rows < 0 || rows > 0x7fffffffLL) return fail(SNICIT_E_INVALID_ARG, "bad rows");
    if (kernel == SNICIT_KERNEL_ELL && !net->has_ell)
        return fail(SNICIT_E_UNSUPPORTED, "network loaded in compact circulant form has no ELL copy");
    if (kernel < 0 || kernel > SNICIT_KERNEL_CIRC_SMEM) return fail(SNICIT_E_INVALID_ARG, "bad kernel");
    if ((kernel == SNICIT_KERNEL_CIRC || kernel == SNICIT_KERNEL_CIRC_SMEM) && net->plan[layer].kind == 0)
        return fail(SNICIT_E_UNSUPPORTED, "layer is not circulant");
    DeviceGuard dg(net->device);
    CUDA_TRY(dg.status);
    CUDA_TRY(ensure_workspace(net, rows, 1, 1));
    CUDA_TRY(launch_iota(net->list0.p, (int)rows, net->counters.p + CNT_LIVE0, net->stream));
    LayerArgs a = layer_args(net, layer, kernel == SNICIT_KERNEL_ELL);
    a.yin = yin;
    a.yout = yout;
    a.rows = net->list0.p;
    a.count = net->counters.p + CNT_LIVE0;
    CUDA_TRY(run_layer(net, layer, kernel, MODE_PLAIN, a, (int)rows));
    CUDA_TRY(cudaStreamSynchronize(net->stream));
    return SNICIT_OK;
}

}  // extern "C"
