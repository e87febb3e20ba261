// avfs_host.cpp -- host runtime behind include/avfs.h.
//
// Native pieces of the flow of Fig. 2:
//   * .bench parser with full-scan DFF cut
//   * levelizer: ASAP levels, gates sorted by level
//   * liveness allocator: interval colouring of waveform buffers over levels
//     (waveform storage dominates); POs / probes are pinned
//   * coefficient store: per-cell blocks, or per-gate blocks with the
//     load capacitance folded in (alpha_i = sum_j beta_ij phi_C(c)^j) when
//     deg_c > 0
//   * simulate driver: stimulus expansion, persistent sweep, overflow reruns
//   * readback (P:L141 step 4)
// Every arithmetic step of the simulation itself runs in avfs_kernels.cu.
#include "avfs.h"

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <unordered_map>
#include <vector>

#include "avfs_internal.h"

using namespace avfs;

namespace {

struct DevBuf {
    void* p = nullptr;
    size_t n = 0;
    DevBuf() = default;
    DevBuf(const DevBuf&) = delete;
    DevBuf& operator=(const DevBuf&) = delete;
    DevBuf(DevBuf&& o) noexcept : p(o.p), n(o.n) { o.p = nullptr; o.n = 0; }
    ~DevBuf() { release(); }
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        n = 0;
    }
    cudaError_t ensure(size_t bytes) {
        if (bytes <= n && p) return cudaSuccess;
        release();
        size_t b = bytes ? bytes : 16;
        cudaError_t e = cudaMalloc(&p, b);
        if (e == cudaSuccess) n = b;
        else p = nullptr;
        return e;
    }
    template <class T> T* as() const { return static_cast<T*>(p); }
};

struct Round {
    int64_t n_sw = 0;
    int64_t sw_first = 0;            // pass 0: contiguous range
    std::vector<int32_t> sws;        // reruns: explicit list
    int32_t capacity = 0, W = 0;
    int64_t region_bytes = 0;
    int32_t grid = 0;
    int64_t spill_want = 0;          // requested heap words (0: no spill heap)
    int64_t spill_words = 0;         // heap words allocated for this round
    int64_t spill_req = 0;           // words requested by the round's gate-warps (incl. failed)
    int32_t grp = 1;                 // slot groups per sweep CTA
    bool spill_exact = false;        // the caller fixed the heap size (options.spill_bytes > 0): no headroom
    int32_t split = 1;               // sweep CTAs per slot group
};

}  // namespace

struct avfs_ctx {
    int dev = -1;
    int n_sm = 0;
    bool sticky = false;
    std::string err;
    cudaStream_t stream = nullptr;

    // library
    bool lib_loaded = false;
    std::vector<std::string> cell_names;
    std::vector<int32_t> cell_nin;
    std::vector<uint16_t> cell_tt;
    int32_t deg_v = 0, deg_c = 0;
    std::vector<double> beta;
    double v_min = 0.55, v_max = 1.1, c_min = 0.5, c_max = 128.0;

    // netlist
    bool net_loaded = false;
    int32_t n_pi = 0, n_gates = 0;
    std::vector<int32_t> gate_cell;
    std::vector<int64_t> fanin_ptr;
    std::vector<int32_t> fanin_sig;
    std::vector<double> d_nom, c_load;
    std::vector<int32_t> po;
    std::unordered_map<std::string, int32_t> names;

    // levelised view
    std::vector<int32_t> level;       // per signal
    std::vector<int32_t> order;       // gates sorted by level
    std::vector<int32_t> level_ptr;   // [depth+1]
    std::vector<int32_t> last_read;   // per signal: max level of a reader, -1 none
    std::vector<int64_t> fanout;      // gate pins reading each signal
    std::vector<uint8_t> is_po;       // per signal
    int32_t depth = 0, kmax = 1, n_dangling = 0;
    std::vector<double> coef;         // coefficient blocks
    std::vector<uint32_t> coef_off;   // per gate: its cell's coefficient block
    std::vector<double> phi_c;        // per gate: phi_C(c_load) (0 when deg_c = 0)

    // plan (options dependent)
    bool plan_valid = false;
    std::vector<uint32_t> loc;        // per signal
    int32_t n_scratch = 0, n_pinned = 0;

    avfs_options opt{};
    std::vector<int32_t> probes;

    std::vector<double> vdd;          // [n_points] first island's supply (sizes by point)
    std::vector<double> vdd_all;      // [n_points][n_isl]
    std::vector<int32_t> island;      // [n_gates] voltage island (NEXT-2)
    int32_t n_isl = 1;
    int64_t n_pairs = 0;
    int32_t words = 0;
    bool stim_set = false;
    int64_t slot_first = 0, slot_count = -1;
    bool pair_mode = false;          // avfs_set_pair_range: pairs [pair_first, + pair_count) at every point
    int64_t pair_first = 0, pair_count = 0;

    // device state
    bool dev_net_valid = false, dev_vdd_valid = false;
    DevBuf d_gates, d_ddesc, d_dtab, d_coef, d_cload, d_island, d_energy, c_loc, c_tclk, c_slot, c_out, d_level_ptr, d_vdd, d_p1, d_p2, d_p1t, d_p2t, d_p1g, d_p2g, d_act, d_latest, d_ovf,
        d_err, d_list[2], d_prev[2], d_pois[2], d_spill_top, d_lvlsync, d_count, d_swround, d_swindex, g_loc, g_init, g_count,
        g_times, g_bad;
    std::vector<DevBuf> arena;        // per round: [buffer][slot group][region]
    std::vector<DevBuf> recs;         // per round: [buffer][slot group] records
    DevBuf d_zero, d_enc;
    std::vector<DevBuf> spill;        // per round: spill heap (kept: readback may point into it)
    int64_t spill_hint = 0;           // heap words the last simulate asked for (all rounds)
    int64_t spill_per_group = 0;      // largest heap words per slot group asked for so far (sizing hint)
    bool spill_known = false;         // spill_per_group measured on this netlist
    int32_t n_batches = 1;            // slot batches of the last simulate (readback keeps the last)
    int32_t* h_pinned = nullptr;      // small pinned host buffer (count, err)
    cudaEvent_t ev0 = nullptr, ev1 = nullptr, ev2 = nullptr, ev3 = nullptr;   // pass-0 sweep; reruns

    // last simulation
    bool sim_done = false, map_valid = false;
    // an asynchronous simulate whose overflow check is still outstanding
    // (settled by avfs_sync or any call that needs the results)
    bool pending = false;
    int pend_r = 0, pend_cur = 0;
    int64_t pend_r0n = 1, pend_hint = 0, pend_slots = 0;
    double pend_sweep_ms = 0;
    std::chrono::steady_clock::time_point pend_t0;
    std::vector<Round> rounds;
    int64_t sim_first = 0, sim_end = 0;
    SlotBox box{};                   // the last simulate's slot box (pair-major slot groups)
    int64_t n_grp = 0;
    avfs_stats stats{};
    DelayParams dparams{};            // delay model of the last simulate (the sweep may evaluate it)
};

static avfs_status finish_pending(avfs_ctx* ctx);   // settles an asynchronous simulate (defined below)

#define SETTLE()                                                                                   \
    do {                                                                                           \
        avfs_status s_ = finish_pending(ctx);                                                      \
        if (s_ != AVFS_OK) return s_;                                                              \
    } while (0)

namespace {

avfs_status fail(avfs_ctx* c, avfs_status st, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    if (c) {
        c->err = buf;
        if (st == AVFS_ERR_CUDA) c->sticky = true;
    }
    return st;
}

#define CK(call)                                                                                   \
    do {                                                                                           \
        cudaError_t e_ = (call);                                                                   \
        if (e_ != cudaSuccess) {                                                                   \
            if (e_ == cudaErrorMemoryAllocation) {                                                 \
                cudaGetLastError();                                                                \
                return fail(ctx, AVFS_ERR_NOMEM, "%s: %s", #call, cudaGetErrorString(e_));         \
            }                                                                                      \
            return fail(ctx, AVFS_ERR_CUDA, "%s: %s", #call, cudaGetErrorString(e_));              \
        }                                                                                          \
    } while (0)

#define CHECK_CTX()                                                                                \
    do {                                                                                           \
        if (!ctx) return AVFS_ERR_ARG;                                                             \
        if (ctx->sticky) return AVFS_ERR_CUDA;                                                     \
        ctx->err.clear();                                                                          \
    } while (0)

bool has_dev(const avfs_ctx* c) { return c->dev >= 0; }

// ---------------------------------------------------------------- levelizer
avfs_status levelize(avfs_ctx* ctx) {
    const int32_t G = ctx->n_gates, S = ctx->n_pi + G;
    ctx->level.assign(S, 0);
    ctx->fanout.assign(S, 0);
    std::vector<int64_t> fo_ptr(S + 1, 0);
    for (int64_t e = 0; e < ctx->fanin_ptr[G]; ++e) fo_ptr[ctx->fanin_sig[e] + 1]++;
    for (int32_t s = 0; s < S; ++s) {
        ctx->fanout[s] = fo_ptr[s + 1];
        fo_ptr[s + 1] += fo_ptr[s];
    }
    std::vector<int32_t> fo_gate(ctx->fanin_ptr[G]);
    {
        std::vector<int64_t> fill(fo_ptr.begin(), fo_ptr.end() - 1);
        for (int32_t g = 0; g < G; ++g)
            for (int64_t e = ctx->fanin_ptr[g]; e < ctx->fanin_ptr[g + 1]; ++e)
                fo_gate[fill[ctx->fanin_sig[e]]++] = g;
    }
    std::vector<int32_t> indeg(G, 0), queue;
    queue.reserve(G);
    for (int32_t g = 0; g < G; ++g) {
        for (int64_t e = ctx->fanin_ptr[g]; e < ctx->fanin_ptr[g + 1]; ++e)
            indeg[g] += ctx->fanin_sig[e] >= ctx->n_pi;
        if (!indeg[g]) queue.push_back(g);
    }
    for (size_t h = 0; h < queue.size(); ++h) {
        const int32_t g = queue[h];
        int32_t lv = 0;
        for (int64_t e = ctx->fanin_ptr[g]; e < ctx->fanin_ptr[g + 1]; ++e)
            lv = std::max(lv, ctx->level[ctx->fanin_sig[e]]);
        ctx->level[ctx->n_pi + g] = lv + 1;
        const int32_t s = ctx->n_pi + g;
        for (int64_t f = fo_ptr[s]; f < fo_ptr[s + 1]; ++f)
            if (--indeg[fo_gate[f]] == 0) queue.push_back(fo_gate[f]);
    }
    if ((int32_t)queue.size() != G) return fail(ctx, AVFS_ERR_PARSE, "netlist has a combinational cycle");
    ctx->depth = 0;
    for (int32_t g = 0; g < G; ++g) ctx->depth = std::max(ctx->depth, ctx->level[ctx->n_pi + g]);
    ctx->order.resize(G);
    for (int32_t g = 0; g < G; ++g) ctx->order[g] = g;
    // by level; within a level, gates with > 2 inputs first, so that they
    // fill the level's first (full, 32-gate) batches and most batches --
    // among them all the small ones at the level's end -- evaluate the
    // 2-input masks only (sweep phase A)
    const bool wide_last = getenv("AVFS_WIDE_LAST") != nullptr && atoi(getenv("AVFS_WIDE_LAST")) != 0;
    std::stable_sort(ctx->order.begin(), ctx->order.end(), [&](int32_t a, int32_t b) {
        const int32_t la = ctx->level[ctx->n_pi + a], lb = ctx->level[ctx->n_pi + b];
        if (la != lb) return la < lb;
        const bool wa = ctx->fanin_ptr[a + 1] - ctx->fanin_ptr[a] > 2, wb = ctx->fanin_ptr[b + 1] - ctx->fanin_ptr[b] > 2;
        return wide_last ? (!wa && wb) : (wa && !wb);
    });
    ctx->level_ptr.assign(ctx->depth + 1, 0);
    for (int32_t g = 0; g < G; ++g) ctx->level_ptr[ctx->level[ctx->n_pi + g]]++;
    for (int32_t L = 1; L <= ctx->depth; ++L) ctx->level_ptr[L] += ctx->level_ptr[L - 1];
    ctx->last_read.assign(S, -1);
    for (int32_t g = 0; g < G; ++g)
        for (int64_t e = ctx->fanin_ptr[g]; e < ctx->fanin_ptr[g + 1]; ++e) {
            int32_t& lr = ctx->last_read[ctx->fanin_sig[e]];
            lr = std::max(lr, ctx->level[ctx->n_pi + g]);
        }
    ctx->is_po.assign(S, 0);
    for (int32_t s : ctx->po) ctx->is_po[s] = 1;
    ctx->n_dangling = 0;
    for (int32_t g = 0; g < G; ++g)
        ctx->n_dangling += (ctx->last_read[ctx->n_pi + g] < 0 && !ctx->is_po[ctx->n_pi + g]);
    ctx->kmax = 1;
    for (int32_t g = 0; g < G; ++g)
        ctx->kmax = std::max<int32_t>(ctx->kmax, (int32_t)(ctx->fanin_ptr[g + 1] - ctx->fanin_ptr[g]));
    return AVFS_OK;
}

// ---------------------------------------------------------------- coefficient store
// The device evaluates Eq. (4) in both variables (NEXT-2): the cells'
// coefficients go to the device unchanged ([cell][pin][pol][deg_v+1][deg_c+1],
// P:L139 "stored in the GPU memory"); per gate only z = phi_C(c_g) is
// precomputed here (P:L117 normalisation of the gate's load).
void build_coef(avfs_ctx* ctx) {
    const size_t nb = (size_t)(ctx->deg_v + 1) * (ctx->deg_c + 1);
    ctx->coef = ctx->beta;
    ctx->coef_off.assign(ctx->n_gates, 0);
    ctx->phi_c.assign(ctx->n_gates, 0.0);
    const double lc0 = std::log2(ctx->c_min), lc1 = std::log2(ctx->c_max);
    for (int32_t g = 0; g < ctx->n_gates; ++g) {
        ctx->coef_off[g] = (uint32_t)((size_t)ctx->gate_cell[g] * 8 * nb);
        if (ctx->deg_c > 0) ctx->phi_c[g] = (std::log2(ctx->c_load[g]) - lc0) / (lc1 - lc0);
    }
}

// ---------------------------------------------------------------- liveness allocator
avfs_status build_plan(avfs_ctx* ctx) {
    if (ctx->plan_valid) return AVFS_OK;
    const int32_t G = ctx->n_gates, S = ctx->n_pi + G;
    std::vector<uint8_t> pinned(S, 0);
    for (int32_t s = ctx->n_pi; s < S; ++s)
        if (ctx->opt.keep_all || ctx->is_po[s]) pinned[s] = 1;
    for (int32_t s : ctx->probes)
        if (s >= ctx->n_pi) pinned[s] = 1;
    ctx->loc.assign(S, 0);
    for (int32_t i = 0; i < ctx->n_pi; ++i) ctx->loc[i] = LOC_PI | (uint32_t)i;
    int32_t np = 0;
    for (int32_t s = ctx->n_pi; s < S; ++s)
        if (pinned[s]) ctx->loc[s] = LOC_PINNED | (uint32_t)np++;
    ctx->n_pinned = np;
    // interval colouring: a buffer written at level L and last read at level R
    // may be rewritten from level max(L, R) + 1 on (the CTA barrier between
    // levels orders the last read before the rewrite).
    std::vector<std::vector<int32_t>> release(ctx->depth + 2);
    std::vector<int32_t> free_list;
    int32_t n_buf = 0;
    for (int32_t L = 1; L <= ctx->depth; ++L) {
        for (int32_t b : release[L]) free_list.push_back(b);
        // the level's gates take the free buffers in ascending order (the
        // smallest last in the vector): consecutive gates of a level mostly
        // get consecutive buffer ids, so their records and regions are adjacent
        if (getenv("AVFS_SORTED_BUFFERS") == nullptr || atoi(getenv("AVFS_SORTED_BUFFERS")) != 0)
            std::sort(free_list.begin(), free_list.end(), std::greater<int32_t>());
        for (int32_t i = ctx->level_ptr[L - 1]; i < ctx->level_ptr[L]; ++i) {
            const int32_t s = ctx->n_pi + ctx->order[i];
            if (pinned[s]) continue;
            int32_t b;
            if (!free_list.empty()) { b = free_list.back(); free_list.pop_back(); }
            else b = n_buf++;
            ctx->loc[s] = LOC_SCRATCH | (uint32_t)b;
            const int32_t until = std::max(L, ctx->last_read[s]);
            release[until + 1].push_back(b);
        }
    }
    ctx->n_scratch = n_buf;
    ctx->plan_valid = true;
    ctx->dev_net_valid = false;
    return AVFS_OK;
}

// arena buffer of a gate output: kept signals first, scratch after (PIs have
// no buffer: their waveforms are the stimulus words, reading C2)
uint32_t buffer_id(const avfs_ctx* ctx, uint32_t loc) {
    const uint32_t kind = loc & LOC_KIND, id = loc & LOC_ID;
    if (kind == LOC_PINNED) return id;
    return (uint32_t)ctx->n_pinned + id;
}

// location code of a gate input as the sweep reads it
uint32_t input_code(const avfs_ctx* ctx, uint32_t loc) {
    if ((loc & LOC_KIND) == LOC_PI) return loc;
    return (loc & LOC_KIND) | buffer_id(ctx, loc);
}

// bytes of one waveform region holding W in-place times (REG_TIMES + 4 W),
// rounded up to AVFS_REGION_ALIGN (default 128: every region -- its entries,
// then its first times -- starts on a cache line, so a reader's entry load
// and the extent prefetch touch the fewest lines; config 4 sweep 65.3 ->
// 61.5 ms for 7 % more arena)
static int64_t region_size(int32_t W) {
    static const int64_t align = [] {
        const char* e = getenv("AVFS_REGION_ALIGN");
        const int64_t a = e ? atoll(e) : 128;
        return a >= 16 ? a : (int64_t)16;
    }();
    const int64_t b = REG_TIMES + 4 * (int64_t)W;
    return (b + align - 1) / align * align;
}

avfs_status upload_netlist(avfs_ctx* ctx) {
    if (ctx->dev_net_valid) return AVFS_OK;
    const int32_t G = ctx->n_gates;
    std::vector<GateDesc> gd(std::max<int32_t>(G, 1));
    std::vector<DelayDesc> dd(std::max<int32_t>(G, 1));
    for (int32_t i = 0; i < G; ++i) {
        const int32_t g = ctx->order[i];
        GateDesc& d = gd[i];
        DelayDesc& e = dd[i];
        std::memset(&d, 0, sizeof d);
        std::memset(&e, 0, sizeof e);
        const int k = (int)(ctx->fanin_ptr[g + 1] - ctx->fanin_ptr[g]);
        for (int p = 0; p < KMAX; ++p) d.in_loc[p] = p < k ? input_code(ctx, ctx->loc[ctx->fanin_sig[ctx->fanin_ptr[g] + p]]) : 0u;
        d.out_loc = buffer_id(ctx, ctx->loc[ctx->n_pi + g]);
        d.sig = (uint32_t)(ctx->n_pi + g);
        const uint32_t ttm = (uint32_t)ctx->cell_tt[ctx->gate_cell[g]] & (0xFFFFu >> (16 - (1 << k)));
        d.ttk = ttm | ((uint32_t)k << 16) | ((ctx->is_po[ctx->n_pi + g] ? 1u : 0u) << 24);
        d.fanout = (uint32_t)std::min<int64_t>(ctx->fanout[ctx->n_pi + g], 0xFFFFFF);
        e.coef_off = ctx->coef_off[g];
        e.z = ctx->phi_c[g];
        e.k = (uint32_t)k;
        e.island = (uint32_t)ctx->island[g];
        for (int p = 0; p < k; ++p)
            for (int pol = 0; pol < 2; ++pol) e.dnom[2 * p + pol] = ctx->d_nom[(ctx->fanin_ptr[g] + p) * 2 + pol];
        for (int p = k; p < KMAX; ++p) e.dnom[2 * p] = e.dnom[2 * p + 1] = 1.0;
    }
    CK(ctx->d_gates.ensure(gd.size() * sizeof(GateDesc)));
    CK(cudaMemcpy(ctx->d_gates.p, gd.data(), gd.size() * sizeof(GateDesc), cudaMemcpyHostToDevice));
    CK(ctx->d_ddesc.ensure(dd.size() * sizeof(DelayDesc)));
    CK(cudaMemcpy(ctx->d_ddesc.p, dd.data(), dd.size() * sizeof(DelayDesc), cudaMemcpyHostToDevice));
    CK(ctx->d_coef.ensure(std::max<size_t>(ctx->coef.size(), 1) * sizeof(double)));
    if (!ctx->coef.empty())
        CK(cudaMemcpy(ctx->d_coef.p, ctx->coef.data(), ctx->coef.size() * sizeof(double), cudaMemcpyHostToDevice));
    CK(ctx->d_island.ensure((size_t)std::max<int32_t>(G, 1) * sizeof(int32_t)));
    CK(cudaMemcpy(ctx->d_island.p, ctx->island.data(), (size_t)G * sizeof(int32_t), cudaMemcpyHostToDevice));
    CK(ctx->d_cload.ensure((size_t)std::max<int32_t>(G, 1) * sizeof(double)));
    CK(cudaMemcpy(ctx->d_cload.p, ctx->c_load.data(), (size_t)G * sizeof(double), cudaMemcpyHostToDevice));
    CK(ctx->d_level_ptr.ensure(ctx->level_ptr.size() * sizeof(int32_t)));
    CK(cudaMemcpy(ctx->d_level_ptr.p, ctx->level_ptr.data(), ctx->level_ptr.size() * sizeof(int32_t),
                  cudaMemcpyHostToDevice));
    ctx->dev_net_valid = true;
    return AVFS_OK;
}

// inputs change: settle an outstanding simulate first (its errors, if any,
// stay in avfs_last_error), then drop its results
void invalidate_sim(avfs_ctx* ctx) {
    if (ctx->pending) {
        const std::string keep = ctx->err;
        if (finish_pending(ctx) == AVFS_OK) ctx->err = keep;
    }
    ctx->sim_done = false;
    ctx->map_valid = false;
}

// ---------------------------------------------------------------- .bench parser
std::string trim(const std::string& s) {
    size_t a = 0, b = s.size();
    while (a < b && isspace((unsigned char)s[a])) ++a;
    while (b > a && isspace((unsigned char)s[b - 1])) --b;
    return s.substr(a, b - a);
}

std::string upper(std::string s) {
    for (auto& ch : s) ch = (char)toupper((unsigned char)ch);
    return s;
}

}  // namespace

// ============================================================================ C-ABI
extern "C" {

const char* avfs_version(void) { return "avfs 0.1 sm_100a"; }

const char* avfs_status_string(avfs_status st) {
    switch (st) {
        case AVFS_OK: return "AVFS_OK";
        case AVFS_ERR_ARG: return "AVFS_ERR_ARG";
        case AVFS_ERR_PARSE: return "AVFS_ERR_PARSE";
        case AVFS_ERR_STATE: return "AVFS_ERR_STATE";
        case AVFS_ERR_CUDA: return "AVFS_ERR_CUDA";
        case AVFS_ERR_NOMEM: return "AVFS_ERR_NOMEM";
        case AVFS_ERR_DELAY_NONPOS: return "AVFS_ERR_DELAY_NONPOS";
        case AVFS_ERR_CAPACITY: return "AVFS_ERR_CAPACITY";
    }
    return "unknown";
}

avfs_status avfs_default_options(avfs_options* o) {
    if (!o) return AVFS_ERR_ARG;
    std::memset(o, 0, sizeof *o);
    o->capacity = 8;
    o->max_rerun_rounds = 3;
    o->warps_per_cta = 8;
    return AVFS_OK;
}

avfs_status avfs_create(int cuda_device, avfs_ctx** out) {
    if (!out) return AVFS_ERR_ARG;
    *out = nullptr;
    avfs_ctx* ctx = new (std::nothrow) avfs_ctx();
    if (!ctx) return AVFS_ERR_NOMEM;
    avfs_default_options(&ctx->opt);
    if (cuda_device >= 0) {
        int n = 0;
        cudaError_t e = cudaGetDeviceCount(&n);
        if (e != cudaSuccess || cuda_device >= n) {
            cudaGetLastError();
            delete ctx;
            return AVFS_ERR_CUDA;
        }
        ctx->dev = cuda_device;
        if (cudaSetDevice(cuda_device) != cudaSuccess ||
            cudaDeviceGetAttribute(&ctx->n_sm, cudaDevAttrMultiProcessorCount, cuda_device) != cudaSuccess ||
            cudaMallocHost(&ctx->h_pinned, 64) != cudaSuccess ||
            cudaEventCreate(&ctx->ev0) != cudaSuccess || cudaEventCreate(&ctx->ev1) != cudaSuccess ||
            cudaEventCreate(&ctx->ev2) != cudaSuccess || cudaEventCreate(&ctx->ev3) != cudaSuccess) {
            cudaGetLastError();
            delete ctx;
            return AVFS_ERR_CUDA;
        }
    }
    *out = ctx;
    return AVFS_OK;
}

void avfs_destroy(avfs_ctx* ctx) {
    if (!ctx) return;
    if (ctx->dev >= 0) {
        cudaSetDevice(ctx->dev);
        if (ctx->h_pinned) cudaFreeHost(ctx->h_pinned);
        if (ctx->ev0) cudaEventDestroy(ctx->ev0);
        if (ctx->ev1) cudaEventDestroy(ctx->ev1);
        if (ctx->ev2) cudaEventDestroy(ctx->ev2);
        if (ctx->ev3) cudaEventDestroy(ctx->ev3);
    }
    delete ctx;
}

const char* avfs_last_error(const avfs_ctx* ctx) { return ctx ? ctx->err.c_str() : "null context"; }

avfs_status avfs_load_library(avfs_ctx* ctx, int32_t n_cells, const avfs_cell* cells, int32_t deg_v,
                              int32_t deg_c, const double* beta, double v_min, double v_max,
                              double c_min_fF, double c_max_fF) {
    CHECK_CTX();
    if (n_cells <= 0 || !cells || !beta) return fail(ctx, AVFS_ERR_ARG, "null library arrays");
    if (deg_v < 0 || deg_v > MAX_DEG || deg_c < 0 || deg_c > MAX_DEG)
        return fail(ctx, AVFS_ERR_ARG, "polynomial degree out of range [0,%d]", MAX_DEG);
    if (!(v_max > v_min) || !(c_max_fF > c_min_fF) || !(c_min_fF > 0))
        return fail(ctx, AVFS_ERR_ARG, "bad normalisation bounds");
    ctx->cell_names.clear();
    ctx->cell_nin.clear();
    ctx->cell_tt.clear();
    for (int32_t c = 0; c < n_cells; ++c) {
        if (cells[c].n_inputs < 1 || cells[c].n_inputs > KMAX)
            return fail(ctx, AVFS_ERR_ARG, "cell %d: n_inputs must be 1..4", c);
        ctx->cell_names.push_back(cells[c].name ? upper(cells[c].name) : std::string());
        ctx->cell_nin.push_back(cells[c].n_inputs);
        ctx->cell_tt.push_back(cells[c].truth_table);
    }
    const size_t nb = (size_t)n_cells * 8 * (deg_v + 1) * (deg_c + 1);
    ctx->beta.assign(beta, beta + nb);
    for (double b : ctx->beta)
        if (!std::isfinite(b)) return fail(ctx, AVFS_ERR_ARG, "non-finite coefficient");
    ctx->deg_v = deg_v;
    ctx->deg_c = deg_c;
    ctx->v_min = v_min;
    ctx->v_max = v_max;
    ctx->c_min = c_min_fF;
    ctx->c_max = c_max_fF;
    ctx->lib_loaded = true;
    ctx->net_loaded = false;
    ctx->stim_set = false;             // stimuli are sized by the netlist's PIs
    ctx->plan_valid = false;
    ctx->dev_net_valid = false;
    invalidate_sim(ctx);
    return AVFS_OK;
}

avfs_status avfs_load_netlist(avfs_ctx* ctx, int32_t n_pi, int32_t n_gates, const int32_t* gate_cell,
                              const int64_t* fanin_ptr, const int32_t* fanin_sig, const double* d_nom_ps,
                              const double* c_load_fF, int32_t n_po, const int32_t* po_sig) {
    CHECK_CTX();
    if (!ctx->lib_loaded) return fail(ctx, AVFS_ERR_STATE, "load the cell library first");
    if (n_pi < 0 || n_gates < 1 || !gate_cell || !fanin_ptr || !fanin_sig || !d_nom_ps || n_po < 0 ||
        (n_po > 0 && !po_sig))
        return fail(ctx, AVFS_ERR_ARG, "bad netlist arrays");
    if (ctx->deg_c > 0 && !c_load_fF) return fail(ctx, AVFS_ERR_ARG, "c_load required when deg_c > 0");
    const int64_t S = (int64_t)n_pi + n_gates;
    if (S >= (int64_t)LOC_ID) return fail(ctx, AVFS_ERR_ARG, "too many signals");
    if (fanin_ptr[0] != 0) return fail(ctx, AVFS_ERR_ARG, "fanin_ptr[0] must be 0");
    for (int32_t g = 0; g < n_gates; ++g) {
        const int64_t k = fanin_ptr[g + 1] - fanin_ptr[g];
        if (gate_cell[g] < 0 || gate_cell[g] >= (int32_t)ctx->cell_nin.size())
            return fail(ctx, AVFS_ERR_ARG, "gate %d: cell index out of range", g);
        if (k != ctx->cell_nin[gate_cell[g]])
            return fail(ctx, AVFS_ERR_ARG, "gate %d: %lld fan-ins for a %d-input cell", g, (long long)k,
                        ctx->cell_nin[gate_cell[g]]);
        for (int64_t e = fanin_ptr[g]; e < fanin_ptr[g + 1]; ++e) {
            if (fanin_sig[e] < 0 || fanin_sig[e] >= S) return fail(ctx, AVFS_ERR_ARG, "gate %d: bad fan-in", g);
            if (fanin_sig[e] == n_pi + g) return fail(ctx, AVFS_ERR_PARSE, "gate %d drives itself", g);
            for (int pol = 0; pol < 2; ++pol)
                if (!(d_nom_ps[2 * e + pol] > 0) || !std::isfinite(d_nom_ps[2 * e + pol]))
                    return fail(ctx, AVFS_ERR_ARG, "gate %d: nominal delay must be finite and > 0", g);
        }
        if (c_load_fF && ctx->deg_c > 0 && !(c_load_fF[g] > 0))
            return fail(ctx, AVFS_ERR_ARG, "gate %d: load must be > 0", g);
    }
    for (int32_t i = 0; i < n_po; ++i)
        if (po_sig[i] < 0 || po_sig[i] >= S) return fail(ctx, AVFS_ERR_ARG, "bad PO signal");
    const int64_t E = fanin_ptr[n_gates];
    ctx->n_pi = n_pi;
    ctx->n_gates = n_gates;
    ctx->gate_cell.assign(gate_cell, gate_cell + n_gates);
    ctx->fanin_ptr.assign(fanin_ptr, fanin_ptr + n_gates + 1);
    ctx->fanin_sig.assign(fanin_sig, fanin_sig + E);
    ctx->d_nom.assign(d_nom_ps, d_nom_ps + 2 * E);
    if (c_load_fF) ctx->c_load.assign(c_load_fF, c_load_fF + n_gates);
    else ctx->c_load.assign(n_gates, 1.0);
    ctx->po.assign(po_sig, po_sig + n_po);
    ctx->island.assign(n_gates, 0);
    if (ctx->n_isl != 1 && !ctx->vdd.empty()) {     // back to one supply per operating point
        ctx->n_isl = 1;
        ctx->vdd_all = ctx->vdd;
        ctx->dev_vdd_valid = false;
    }
    ctx->net_loaded = false;
    avfs_status st = levelize(ctx);
    if (st != AVFS_OK) return st;
    build_coef(ctx);
    ctx->net_loaded = true;
    ctx->stim_set = false;             // stimuli were packed for the previous netlist's PIs
    ctx->spill_per_group = 0;          // the heap sizing hint belongs to the previous netlist
    ctx->spill_known = false;
    ctx->spill_hint = 0;
    ctx->plan_valid = false;
    ctx->dev_net_valid = false;
    ctx->names.clear();
    invalidate_sim(ctx);
    return AVFS_OK;
}

avfs_status avfs_load_bench(avfs_ctx* ctx, const char* text, size_t len, const double* d_nom_ps,
                            const double* c_load_fF) {
    CHECK_CTX();
    if (!ctx->lib_loaded) return fail(ctx, AVFS_ERR_STATE, "load the cell library first");
    if (!text || !d_nom_ps) return fail(ctx, AVFS_ERR_ARG, "null text or delays");
    std::vector<std::string> inputs, outputs, dff_q, dff_d;
    struct GateLine { std::string out, type; std::vector<std::string> ins; int line; };
    std::vector<GateLine> gates;
    std::string src(text, len);
    size_t pos = 0;
    int lineno = 0;
    while (pos <= src.size()) {
        size_t nl = src.find('\n', pos);
        if (nl == std::string::npos) nl = src.size();
        std::string line = src.substr(pos, nl - pos);
        pos = nl + 1;
        ++lineno;
        const size_t hash = line.find('#');
        if (hash != std::string::npos) line = line.substr(0, hash);
        line = trim(line);
        if (line.empty()) continue;
        const size_t lp = line.find('('), rp = line.rfind(')');
        if (lp == std::string::npos || rp == std::string::npos || rp < lp)
            return fail(ctx, AVFS_ERR_PARSE, "line %d: expected '(' ... ')'", lineno);
        const size_t eq = line.find('=');
        if (eq == std::string::npos || eq > lp) {
            const std::string kw = upper(trim(line.substr(0, lp)));
            const std::string arg = trim(line.substr(lp + 1, rp - lp - 1));
            if (kw == "INPUT") inputs.push_back(arg);
            else if (kw == "OUTPUT") outputs.push_back(arg);
            else return fail(ctx, AVFS_ERR_PARSE, "line %d: unknown keyword '%s'", lineno, kw.c_str());
            continue;
        }
        GateLine g;
        g.line = lineno;
        g.out = trim(line.substr(0, eq));
        g.type = upper(trim(line.substr(eq + 1, lp - eq - 1)));
        std::string args = line.substr(lp + 1, rp - lp - 1);
        size_t a = 0;
        while (a <= args.size()) {
            size_t comma = args.find(',', a);
            if (comma == std::string::npos) comma = args.size();
            std::string t = trim(args.substr(a, comma - a));
            if (!t.empty()) g.ins.push_back(t);
            a = comma + 1;
        }
        if (g.out.empty() || g.ins.empty()) return fail(ctx, AVFS_ERR_PARSE, "line %d: malformed gate", lineno);
        if (g.type == "DFF") {
            if (g.ins.size() != 1) return fail(ctx, AVFS_ERR_PARSE, "line %d: DFF takes one input", lineno);
            dff_q.push_back(g.out);
            dff_d.push_back(g.ins[0]);
        } else {
            gates.push_back(g);
        }
    }
    std::unordered_map<std::string, int32_t> id;
    int32_t n_pi = 0;
    for (auto& s : inputs) {
        if (id.count(s)) return fail(ctx, AVFS_ERR_PARSE, "duplicate input '%s'", s.c_str());
        id[s] = n_pi++;
    }
    for (auto& s : dff_q) {    // full-scan cut: DFF outputs become pseudo PIs
        if (id.count(s)) return fail(ctx, AVFS_ERR_PARSE, "duplicate net '%s'", s.c_str());
        id[s] = n_pi++;
    }
    const int32_t G = (int32_t)gates.size();
    for (int32_t g = 0; g < G; ++g) {
        if (id.count(gates[g].out)) return fail(ctx, AVFS_ERR_PARSE, "line %d: net '%s' driven twice", gates[g].line, gates[g].out.c_str());
        id[gates[g].out] = n_pi + g;
    }
    std::vector<int32_t> cell(G), fsig;
    std::vector<int64_t> fptr(G + 1, 0);
    for (int32_t g = 0; g < G; ++g) {
        const int k = (int)gates[g].ins.size();
        std::string want = gates[g].type + std::to_string(k);
        std::vector<std::string> cands = {want, gates[g].type};
        if (k == 1) {
            if (gates[g].type == "NOT" || gates[g].type == "INV") cands = {"INV", "NOT"};
            if (gates[g].type == "BUFF" || gates[g].type == "BUF") cands = {"BUF", "BUFF"};
        }
        int32_t ci = -1;
        for (auto& cn : cands) {
            for (size_t c = 0; c < ctx->cell_names.size() && ci < 0; ++c)
                if (ctx->cell_names[c] == cn && ctx->cell_nin[c] == k) ci = (int32_t)c;
            if (ci >= 0) break;
        }
        if (ci < 0) return fail(ctx, AVFS_ERR_PARSE, "line %d: no %d-input library cell for '%s'", gates[g].line, k, gates[g].type.c_str());
        cell[g] = ci;
        for (auto& s : gates[g].ins) {
            auto it = id.find(s);
            if (it == id.end()) return fail(ctx, AVFS_ERR_PARSE, "line %d: undriven net '%s'", gates[g].line, s.c_str());
            fsig.push_back(it->second);
        }
        fptr[g + 1] = (int64_t)fsig.size();
    }
    std::vector<int32_t> po;
    for (auto& s : outputs) {
        auto it = id.find(s);
        if (it == id.end()) return fail(ctx, AVFS_ERR_PARSE, "undriven output '%s'", s.c_str());
        po.push_back(it->second);
    }
    for (auto& s : dff_d) {    // DFF inputs become pseudo POs
        auto it = id.find(s);
        if (it == id.end()) return fail(ctx, AVFS_ERR_PARSE, "undriven DFF input '%s'", s.c_str());
        po.push_back(it->second);
    }
    avfs_status st = avfs_load_netlist(ctx, n_pi, G, cell.data(), fptr.data(), fsig.data(), d_nom_ps, c_load_fF,
                                       (int32_t)po.size(), po.data());
    if (st != AVFS_OK) return st;
    ctx->names = std::move(id);
    return AVFS_OK;
}

avfs_status avfs_find_signal(avfs_ctx* ctx, const char* name, int32_t* sig) {
    CHECK_CTX();
    if (!name || !sig) return fail(ctx, AVFS_ERR_ARG, "null argument");
    auto it = ctx->names.find(name);
    if (it == ctx->names.end()) return fail(ctx, AVFS_ERR_ARG, "no net named '%s'", name);
    *sig = it->second;
    return AVFS_OK;
}

avfs_status avfs_get_netlist_info(avfs_ctx* ctx, avfs_netlist_info* info) {
    CHECK_CTX();
    if (!info) return fail(ctx, AVFS_ERR_ARG, "null info");
    if (!ctx->net_loaded) return fail(ctx, AVFS_ERR_STATE, "no netlist");
    avfs_status st = build_plan(ctx);
    if (st != AVFS_OK) return st;
    info->n_pi = ctx->n_pi;
    info->n_gates = ctx->n_gates;
    info->n_po = (int32_t)ctx->po.size();
    info->depth = ctx->depth;
    info->max_fanin = ctx->kmax;
    info->n_scratch_buffers = ctx->n_scratch;
    info->n_pinned = ctx->n_pinned;
    info->n_dangling = ctx->n_dangling;
    info->n_edges = ctx->fanin_ptr[ctx->n_gates];
    return AVFS_OK;
}

avfs_status avfs_get_levels(avfs_ctx* ctx, int32_t* level) {
    CHECK_CTX();
    if (!level) return fail(ctx, AVFS_ERR_ARG, "null output");
    if (!ctx->net_loaded) return fail(ctx, AVFS_ERR_STATE, "no netlist");
    std::copy(ctx->level.begin(), ctx->level.end(), level);
    return AVFS_OK;
}

avfs_status avfs_get_buffer_map(avfs_ctx* ctx, int32_t* out) {
    CHECK_CTX();
    if (!out) return fail(ctx, AVFS_ERR_ARG, "null output");
    if (!ctx->net_loaded) return fail(ctx, AVFS_ERR_STATE, "no netlist");
    avfs_status st = build_plan(ctx);
    if (st != AVFS_OK) return st;
    for (size_t s = 0; s < ctx->loc.size(); ++s) {
        const uint32_t l = ctx->loc[s];
        const uint32_t kind = l & LOC_KIND;
        out[s] = kind == LOC_PI ? -1 : kind == LOC_SCRATCH ? (int32_t)(l & LOC_ID) : -2 - (int32_t)(l & LOC_ID);
    }
    return AVFS_OK;
}

static avfs_status set_points(avfs_ctx* ctx, int32_t n_isl, const int32_t* island, int32_t n_points,
                              const double* vdd) {
    if (n_points < 1 || n_isl < 1 || !vdd) return fail(ctx, AVFS_ERR_ARG, "need at least one operating point / island");
    for (int64_t k = 0; k < (int64_t)n_points * n_isl; ++k)
        if (!std::isfinite(vdd[k])) return fail(ctx, AVFS_ERR_ARG, "non-finite Vdd");
    if (island) {
        if (!ctx->net_loaded) return fail(ctx, AVFS_ERR_STATE, "load a netlist before assigning islands");
        for (int32_t g = 0; g < ctx->n_gates; ++g)
            if (island[g] < 0 || island[g] >= n_isl) return fail(ctx, AVFS_ERR_ARG, "gate %d: island out of range", g);
        ctx->island.assign(island, island + ctx->n_gates);
    } else if (ctx->net_loaded) {
        ctx->island.assign(ctx->n_gates, 0);
    }
    ctx->n_isl = n_isl;
    ctx->vdd_all.assign(vdd, vdd + (size_t)n_points * n_isl);
    ctx->vdd.resize(n_points);
    for (int32_t k = 0; k < n_points; ++k) ctx->vdd[k] = vdd[(size_t)k * n_isl];
    ctx->dev_vdd_valid = false;
    ctx->dev_net_valid = false;          // island index lives in the delay descriptors
    invalidate_sim(ctx);
    return AVFS_OK;
}

avfs_status avfs_set_operating_points(avfs_ctx* ctx, int32_t n_vdd, const double* vdd) {
    CHECK_CTX();
    return set_points(ctx, 1, nullptr, n_vdd, vdd);
}

avfs_status avfs_set_voltage_islands(avfs_ctx* ctx, int32_t n_islands, const int32_t* island_of_gate,
                                     int32_t n_points, const double* vdd_volts) {
    CHECK_CTX();
    return set_points(ctx, n_islands, island_of_gate, n_points, vdd_volts);
}

avfs_status avfs_set_stimuli(avfs_ctx* ctx, int64_t n_pairs, const uint32_t* p1, const uint32_t* p2,
                             int32_t is_device) {
    CHECK_CTX();
    if (!ctx->net_loaded) return fail(ctx, AVFS_ERR_STATE, "load a netlist first");
    if (n_pairs < 1 || !p1 || !p2) return fail(ctx, AVFS_ERR_ARG, "bad stimuli");
    if (!has_dev(ctx)) return fail(ctx, AVFS_ERR_STATE, "host-only context");
    const int32_t words = (ctx->n_pi + 31) / 32;
    const size_t bytes = (size_t)n_pairs * std::max(words, 1) * sizeof(uint32_t);
    CK(cudaSetDevice(ctx->dev));
    CK(ctx->d_p1.ensure(bytes));
    CK(ctx->d_p2.ensure(bytes));
    if (words > 0) {
        const cudaMemcpyKind kind = is_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
        CK(cudaMemcpyAsync(ctx->d_p1.p, p1, (size_t)n_pairs * words * 4, kind, ctx->stream));
        CK(cudaMemcpyAsync(ctx->d_p2.p, p2, (size_t)n_pairs * words * 4, kind, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
    }
    ctx->n_pairs = n_pairs;
    ctx->words = words;
    ctx->stim_set = true;
    invalidate_sim(ctx);
    return AVFS_OK;
}

avfs_status avfs_set_slot_range(avfs_ctx* ctx, int64_t first_slot, int64_t n_slots) {
    CHECK_CTX();
    if (first_slot < 0) return fail(ctx, AVFS_ERR_ARG, "negative first slot");
    ctx->slot_first = first_slot;
    ctx->slot_count = n_slots;
    ctx->pair_mode = false;
    invalidate_sim(ctx);
    return AVFS_OK;
}

avfs_status avfs_set_pair_range(avfs_ctx* ctx, int64_t first_pair, int64_t n_pairs) {
    CHECK_CTX();
    if (first_pair < 0 || n_pairs < 1) return fail(ctx, AVFS_ERR_ARG, "bad pair range [%lld, +%lld)",
                                                    (long long)first_pair, (long long)n_pairs);
    ctx->pair_mode = true;
    ctx->pair_first = first_pair;
    ctx->pair_count = n_pairs;
    ctx->slot_first = 0;
    ctx->slot_count = -1;
    invalidate_sim(ctx);
    return AVFS_OK;
}

avfs_status avfs_set_options(avfs_ctx* ctx, const avfs_options* o) {
    CHECK_CTX();
    if (!o) return fail(ctx, AVFS_ERR_ARG, "null options");
    if (o->capacity < 1 || o->capacity > 1024) return fail(ctx, AVFS_ERR_ARG, "capacity must be in [1, 1024]");
    if (o->quantum_ps < 0 || !std::isfinite(o->quantum_ps)) return fail(ctx, AVFS_ERR_ARG, "bad quantum");
    if (o->n_probe < 0 || (o->n_probe > 0 && !o->probe_sig)) return fail(ctx, AVFS_ERR_ARG, "bad probes");
    if (o->warps_per_cta < 0 || o->warps_per_cta > 32) return fail(ctx, AVFS_ERR_ARG, "warps_per_cta in [0,32]");
    if (o->max_rerun_rounds < 0 || o->max_rerun_rounds > 6) return fail(ctx, AVFS_ERR_ARG, "max_rerun_rounds in [0,6]");
    std::vector<int32_t> pr(o->probe_sig, o->probe_sig + o->n_probe);
    if (ctx->net_loaded)
        for (int32_t s : pr)
            if (s < 0 || s >= ctx->n_pi + ctx->n_gates) return fail(ctx, AVFS_ERR_ARG, "probe %d out of range", s);
    const bool plan_change = !ctx->plan_valid || o->keep_all != ctx->opt.keep_all || pr != ctx->probes;
    ctx->opt = *o;
    ctx->opt.probe_sig = nullptr;
    ctx->probes = pr;
    if (plan_change) ctx->plan_valid = false;
    invalidate_sim(ctx);
    return AVFS_OK;
}

avfs_status avfs_sync(avfs_ctx* ctx) {
    CHECK_CTX();
    if (!has_dev(ctx)) return AVFS_OK;
    SETTLE();
    CK(cudaStreamSynchronize(ctx->stream));
    return AVFS_OK;
}

static void release_rerun_memory(avfs_ctx* ctx) {
    for (size_t r = 1; r < ctx->arena.size(); ++r) ctx->arena[r].release();
    for (size_t r = 1; r < ctx->recs.size(); ++r) ctx->recs[r].release();
    for (size_t r = 1; r < ctx->spill.size(); ++r) ctx->spill[r].release();
}

static avfs_status run_round(avfs_ctx* ctx, Round& R, int round_idx, const int32_t* d_sw_list,
                             const int32_t* d_prev_idx, bool timed) {
    const bool rerun = round_idx > 0;
    const int wmax = AVFS_SWEEP_THREADS / 32;
    int wpc = ctx->opt.warps_per_cta > 0 ? ctx->opt.warps_per_cta : wmax;
    wpc = std::min(wpc, wmax);
    const double per_level = ctx->depth > 0 ? (double)ctx->n_gates / ctx->depth : 1.0;
    // slot groups per sweep CTA: two by default (each group has its own
    // level barrier, so one group's wait overlaps the other's work); more
    // for narrow netlists (few gates per level), up to 8, until every warp
    // has two batches (2 x 32 gates) of a level; one if the groups would not
    // fill the SMs
    int grp = wpc >= 2 ? 2 : 1;
    while (grp < std::min(wpc, 8) && per_level / (double)(wpc / grp) < 64.0) grp *= 2;
    const int smem = sweep_smem_bytes(wpc, grp);
    int bps = 0;
    CK(sweep_occupancy(wpc, smem, &bps));
    if (bps < 1) return fail(ctx, AVFS_ERR_CAPACITY, "sweep kernel does not fit on an SM (smem %d)", smem);
    const int64_t resident = (int64_t)ctx->n_sm * bps;
    if (grp == 2 && R.n_sw < 2 * resident) grp = 1;            // too few groups to pair
    if (const char* e = getenv("AVFS_GROUPS_PER_CTA")) grp = std::max(1, std::min(wpc, atoi(e)));
    while (wpc % grp) grp /= 2;
    // few slot groups for the SMs (last wave mostly empty, e.g. reruns): S
    // co-resident CTAs share a group; S minimises waves / S, with 5 % per
    // doubling of S for the cross-CTA level barriers, ties to the smaller S,
    // and every warp keeps >= 2 gates of a level
    int split = 1;
    if (grp == 1) {
        double best = 1e300;
        for (int S = 1, lg = 0; S <= 16; S *= 2, ++lg) {
            if (S > 1 && per_level / S / wpc < 2.0) break;
            const int64_t g = std::max<int64_t>(resident / S * S, S);
            const double cost = (double)((R.n_sw * S + g - 1) / g) / S * (1.0 + 0.05 * lg);
            if (cost < best - 1e-9) { best = cost; split = S; }
        }
        if (const char* e = getenv("AVFS_SPLIT")) split = std::max(1, std::min(16, atoi(e)));
    }
    R.grp = grp;
    R.split = split;
    if (split > 1) {
        const int64_t items = R.n_sw * split;
        R.grid = (int32_t)std::min<int64_t>(items, std::max<int64_t>(resident / split * split, split));
    } else {
        R.grid = (int32_t)std::min<int64_t>((R.n_sw + grp - 1) / grp, resident);
    }
    if (R.grid < 1) R.grid = 1;
    if ((int)ctx->arena.size() <= round_idx) ctx->arena.resize(round_idx + 1);
    if ((int)ctx->recs.size() <= round_idx) ctx->recs.resize(round_idx + 1);
    const int64_t n_buf = (int64_t)ctx->n_pinned + ctx->n_scratch;
    if ((uint64_t)R.n_sw * R.region_bytes >= (1ull << 32))
        return fail(ctx, AVFS_ERR_NOMEM, "slot-group stride exceeds 4 GiB; restrict the slot range");
    {
        const size_t bytes = (size_t)std::max<int64_t>(n_buf, 1) * R.n_sw * R.region_bytes;
        cudaError_t e = ctx->arena[round_idx].ensure(bytes);
        if (e == cudaErrorMemoryAllocation && round_idx == 0) {   // retained rerun memory: give it back
            cudaGetLastError();
            release_rerun_memory(ctx);
            e = ctx->arena[round_idx].ensure(bytes);
        }
        CK(e);
    }
    CK(ctx->recs[round_idx].ensure((size_t)std::max<int64_t>(n_buf, 1) * R.n_sw * sizeof(uint4)));
    CK(ctx->d_ovf.ensure(std::max<int64_t>(R.n_sw, 1) * sizeof(int32_t)));
    CK(cudaMemsetAsync(ctx->d_ovf.p, 0, R.n_sw * sizeof(int32_t), ctx->stream));
    // spill heap: the requested size, within free device memory (keep 1 GiB)
    if ((int)ctx->spill.size() <= round_idx) ctx->spill.resize(round_idx + 1);
    R.spill_words = 0;
    if (R.spill_want > 0 && ctx->spill[round_idx].n >= (size_t)R.spill_want * 4) {
        R.spill_words = (int64_t)(ctx->spill[round_idx].n / 4);     // reuse the heap (with its headroom)
        if (R.spill_exact) R.spill_words = R.spill_want;
    } else if (R.spill_want > 0) {
        if (round_idx == 0) release_rerun_memory(ctx);   // pass 0's heap grows: retained rerun memory goes first
        size_t fr = 0, tot = 0;
        CK(cudaMemGetInfo(&fr, &tot));
        const size_t have = ctx->spill[round_idx].n;
        // keep 1 GiB, and for a rerun room for one more rerun round's arena
        const size_t keep = (1ull << 30) + (round_idx > 0 ? ctx->arena[round_idx].n + ctx->recs[round_idx].n : 0);
        const size_t avail = fr + have > keep ? fr + have - keep : 0;
        // 25 % headroom so that slowly growing requests do not reallocate every run
        size_t bytes = std::min<size_t>((size_t)R.spill_want * (R.spill_exact ? 4 : 5), avail) & ~(size_t)15;
        while (bytes >= 16 && ctx->spill[round_idx].ensure(bytes) != cudaSuccess) {
            cudaGetLastError();
            bytes = (bytes / 2) & ~(size_t)15;
        }
        if (bytes >= 16) R.spill_words = (int64_t)(bytes / 4);
    }
    CK(ctx->d_spill_top.ensure(8 * 8));
    CK(cudaMemsetAsync(ctx->d_spill_top.as<unsigned long long>() + round_idx, 0, 8, ctx->stream));
    const size_t pois_words = ((size_t)std::max<int64_t>(R.n_sw, 1) * std::max(ctx->n_gates, 1) + 31) / 32;
    DevBuf& pois = ctx->d_pois[round_idx & 1];
    CK(pois.ensure(pois_words * 4));
    CK(cudaMemsetAsync(pois.p, 0, pois_words * 4, ctx->stream));
    if (ctx->d_zero.n < 16 + 128) {                 // 4 zero times, then 32 PI entries {n = 1, offset 0}
        CK(ctx->d_zero.ensure(16 + 128));
        uint32_t init[36] = {0u, 0u, 0u, 0u};
        for (int k = 4; k < 36; ++k) init[k] = 1u;
        CK(cudaMemcpy(ctx->d_zero.p, init, sizeof init, cudaMemcpyHostToDevice));
    }
    SweepParams p{};
    p.gates = ctx->d_gates.as<GateDesc>();
    p.level_ptr = ctx->d_level_ptr.as<int32_t>();
    p.depth = ctx->depth;
    p.n_gates = ctx->n_gates;
    p.dtab = ctx->opt.delay_in_sweep ? nullptr : ctx->d_dtab.as<float>();
    p.dp = ctx->dparams;
    p.p1g = ctx->d_p1g.as<uint32_t>();
    p.p2g = ctx->d_p2g.as<uint32_t>();
    p.n_grp = ctx->n_grp;
    p.box = ctx->box;
    p.n_vdd = (int32_t)ctx->vdd.size();
    p.sw_list = d_sw_list;
    p.sw_first = R.sw_first;
    p.n_sw = R.n_sw;
    p.i_base = 0;
    p.pin_n_sw = R.n_sw;
    p.arena = ctx->arena[round_idx].as<uint8_t>();
    p.region_bytes = R.region_bytes;
    p.recs = ctx->recs[round_idx].as<uint4>();
    p.n_buf = n_buf;
    p.W = R.W;
    p.grp_per_cta = R.grp;
    p.split = R.split;
    if (R.split > 1) {
        CK(ctx->d_lvlsync.ensure((size_t)R.n_sw * 4));
        CK(cudaMemsetAsync(ctx->d_lvlsync.p, 0, (size_t)R.n_sw * 4, ctx->stream));
        p.lvl_sync = ctx->d_lvlsync.as<unsigned int>();
    }
    p.n_pi = ctx->n_pi;
    p.spill = ctx->spill[round_idx].as<float>();
    p.spill_top = ctx->d_spill_top.as<unsigned long long>() + round_idx;
    p.spill_words = (uint64_t)R.spill_words;
    p.pois = pois.as<uint32_t>();
    p.pois_prev = round_idx == 0 ? nullptr : ctx->d_pois[(round_idx - 1) & 1].as<uint32_t>();
    p.prev_idx = d_prev_idx;
    p.zero = ctx->d_zero.as<float>();
    p.pi_ents = reinterpret_cast<const uint32_t*>(ctx->d_zero.as<uint8_t>() + 16);
    p.act = ctx->d_act.as<unsigned long long>();
    p.latest = ctx->d_latest.as<unsigned int>();
    p.ovf = ctx->d_ovf.as<int32_t>();
    p.enc_units = ctx->d_enc.as<unsigned long long>();
    if (timed) CK(cudaEventRecord(ctx->ev0, ctx->stream));
    CK(launch_sweep(p, rerun, R.grid, wpc, ctx->stream));
    ctx->stats.launches++;
    if (timed) CK(cudaEventRecord(ctx->ev1, ctx->stream));
    if (round_idx == 0) ctx->stats.warps_per_cta = wpc;
    return AVFS_OK;
}

}  // extern "C"

// Overflow check of the last round: compaction of the overflowed slot groups
// and asynchronous copies of their count, the delay error flag and the
// round's heap request into pinned host memory.
static avfs_status issue_checks(avfs_ctx* ctx, int r, int cur) {
    Round& prev = ctx->rounds.back();
    CK(ctx->d_list[cur].ensure(std::max<int64_t>(prev.n_sw, 1) * sizeof(int32_t)));
    CK(ctx->d_prev[cur].ensure(std::max<int64_t>(prev.n_sw, 1) * sizeof(int32_t)));
    CK(cudaMemsetAsync(ctx->d_count.p, 0, 16, ctx->stream));
    CK(launch_compact_overflow(ctx->d_ovf.as<int32_t>(), prev.n_sw,
                               r == 0 ? nullptr : ctx->d_list[cur ^ 1].as<int32_t>(), prev.sw_first,
                               ctx->d_list[cur].as<int32_t>(), ctx->d_prev[cur].as<int32_t>(),
                               ctx->d_count.as<int32_t>(), ctx->stream));
    ctx->stats.launches++;
    CK(cudaMemcpyAsync(ctx->h_pinned, ctx->d_count.p, 4, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaMemcpyAsync(ctx->h_pinned + 1, ctx->d_err.p, 4, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaMemcpyAsync(ctx->h_pinned + 2, ctx->d_spill_top.as<unsigned long long>() + r, 8,
                       cudaMemcpyDeviceToHost, ctx->stream));
    return AVFS_OK;
}

// Wait for the outstanding overflow check of the current batch; rerun the
// overflowed slot groups (H7) until none is left, then fold the batch's heap
// requests into the sizing hints.
static avfs_status settle_batch(avfs_ctx* ctx) {
    avfs_status st = AVFS_OK;
    for (;;) {
        const int r = ctx->pend_r;
        const int cur = ctx->pend_cur;
        Round& prev = ctx->rounds.back();
        CK(cudaStreamSynchronize(ctx->stream));
        {
            unsigned long long req = 0;
            std::memcpy(&req, ctx->h_pinned + 2, 8);
            prev.spill_req = (int64_t)req;
            ctx->stats.spill_bytes += 4 * std::min<int64_t>(prev.spill_req, prev.spill_words);
            ctx->stats.spill_heap_bytes += 4 * prev.spill_words;
        }
        if (ctx->h_pinned[1] & 1)
            return fail(ctx, AVFS_ERR_DELAY_NONPOS, "a delay d' = d_nom (1 + f(P)) evaluated to <= 0");
        const int32_t n_ovf = ctx->h_pinned[0];
        if (getenv("AVFS_DEBUG"))
            fprintf(stderr, "[avfs] round %d: %d overflowed groups, heap %.2f GB, requested %.2f GB\n", r, n_ovf,
                    4e-9 * (double)prev.spill_words, 4e-9 * (double)prev.spill_req);
        if (n_ovf == 0) break;
        if (r >= ctx->opt.max_rerun_rounds)
            return fail(ctx, AVFS_ERR_CAPACITY, "%d slot groups still overflow at capacity %d after %d reruns",
                        n_ovf, prev.capacity, r);
        Round Rn;
        Rn.n_sw = n_ovf;
        Rn.sws.resize(n_ovf);
        CK(cudaMemcpy(Rn.sws.data(), ctx->d_list[cur].p, n_ovf * sizeof(int32_t), cudaMemcpyDeviceToHost));
        // with a spill heap the overflow was heap exhaustion: same capacity, a
        // heap 4x what was asked for (poisoned cones asked for nothing), at
        // least 64 MiB; without one, 4x capacity
        if (prev.spill_want > 0) {
            Rn.capacity = prev.capacity;
            int64_t floor_words = (64ll << 20) / 4;
            if (const char* e = getenv("AVFS_RERUN_HEAP_MIN_BYTES")) floor_words = std::max<int64_t>(16, atoll(e) / 4);
            Rn.spill_want = std::max<int64_t>(4 * std::max<int64_t>(prev.spill_req, prev.spill_words), floor_words);
        } else {
            Rn.capacity = std::min(prev.capacity * 4, 1024);
        }
        Rn.W = 32 * Rn.capacity;
        Rn.region_bytes = region_size(Rn.W);
        ctx->stats.overflow_slot_warps += n_ovf;
        ctx->stats.rerun_rounds++;
        if (ctx->opt.profile && r == 0) CK(cudaEventRecord(ctx->ev2, ctx->stream));
        st = run_round(ctx, Rn, r + 1, ctx->d_list[cur].as<int32_t>(), ctx->d_prev[cur].as<int32_t>(), false);
        if (st != AVFS_OK) return st;
        if (ctx->opt.profile) CK(cudaEventRecord(ctx->ev3, ctx->stream));
        ctx->rounds.push_back(std::move(Rn));
        ctx->pend_r = r + 1;
        ctx->pend_cur = cur ^ 1;
        st = issue_checks(ctx, ctx->pend_r, ctx->pend_cur);
        if (st != AVFS_OK) return st;
    }
    int64_t req = 0;
    for (const Round& R : ctx->rounds) req += R.spill_req;
    ctx->pend_hint = std::max(ctx->pend_hint, req);
    ctx->spill_per_group = std::max<int64_t>(ctx->spill_per_group, (req + ctx->pend_r0n - 1) / ctx->pend_r0n);
    ctx->spill_known = true;
    if (ctx->opt.profile) {
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, ctx->ev0, ctx->ev1));
        ctx->pend_sweep_ms += ms;
        if (ctx->pend_r > 0) {                          // this batch reran: time of its rerun rounds
            CK(cudaEventElapsedTime(&ms, ctx->ev2, ctx->ev3));
            ctx->stats.rerun_ms += ms;
        }
    }
    return AVFS_OK;
}

// Settle an asynchronous simulate (avfs_sync, and every call that reads its
// results): overflow reruns, errors, statistics.
static avfs_status finish_pending(avfs_ctx* ctx) {
    if (!ctx->pending) return AVFS_OK;
    ctx->pending = false;
    avfs_status st = settle_batch(ctx);
    if (st != AVFS_OK) return st;
    ctx->spill_hint = ctx->pend_hint;
    if (ctx->opt.profile) ctx->stats.sweep_ms = ctx->pend_sweep_ms;
    ctx->stats.batches = ctx->n_batches;
    int64_t ab = 0;
    for (size_t r = 0; r < ctx->rounds.size(); ++r) ab += (int64_t)ctx->arena[r].n;
    ctx->stats.arena_bytes = ab;
    ctx->stats.sim_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - ctx->pend_t0).count();
    ctx->sim_done = true;
    return AVFS_OK;
}

extern "C" {

avfs_status avfs_simulate(avfs_ctx* ctx, void* cuda_stream) {
    CHECK_CTX();
    if (!has_dev(ctx)) return fail(ctx, AVFS_ERR_STATE, "host-only context");
    if (!ctx->net_loaded || !ctx->stim_set || ctx->vdd.empty())
        return fail(ctx, AVFS_ERR_STATE, "netlist, stimuli and operating points must be set");
    // the sweep forms activity rows (signal x points) and delay-table rows
    // (gate x 4 pins x points) as 32-bit element offsets
    if ((int64_t)(ctx->n_pi + ctx->n_gates) * (int64_t)ctx->vdd.size() >= (int64_t(1) << 32) ||
        (int64_t)ctx->n_gates * 4 * (int64_t)ctx->vdd.size() >= (int64_t(1) << 32))
        return fail(ctx, AVFS_ERR_ARG, "signals x operating points too large for 32-bit row offsets");
    SETTLE();                                          // a previous simulate's reruns (same stream)
    const auto t0 = std::chrono::steady_clock::now();
    CK(cudaSetDevice(ctx->dev));
    ctx->stream = static_cast<cudaStream_t>(cuda_stream);
    avfs_status st = build_plan(ctx);
    if (st != AVFS_OK) return st;
    st = upload_netlist(ctx);
    if (st != AVFS_OK) return st;
    if (!ctx->dev_vdd_valid) {
        CK(ctx->d_vdd.ensure(ctx->vdd_all.size() * sizeof(double)));
        CK(cudaMemcpy(ctx->d_vdd.p, ctx->vdd_all.data(), ctx->vdd_all.size() * sizeof(double), cudaMemcpyHostToDevice));
        ctx->dev_vdd_valid = true;
    }
    invalidate_sim(ctx);
    const int64_t P = ctx->n_pairs;
    const int32_t V = (int32_t)ctx->vdd.size();
    const int64_t total = P * V;
    const int64_t first = ctx->slot_first;
    const int64_t end = ctx->slot_count < 0 ? total : std::min(total, first + ctx->slot_count);
    if (first >= end) return fail(ctx, AVFS_ERR_ARG, "empty slot range [%lld, %lld)", (long long)first, (long long)end);
    if (ctx->pair_mode && ctx->pair_first + ctx->pair_count > P)
        return fail(ctx, AVFS_ERR_ARG, "pair range [%lld, %lld) beyond the %lld stimulus pairs",
                    (long long)ctx->pair_first, (long long)(ctx->pair_first + ctx->pair_count), (long long)P);
    ctx->sim_first = first;
    ctx->sim_end = end;
    const int32_t n_pw = (int32_t)((P + 31) / 32);
    // the slot box (SlotBox): the pairs and operating points the range
    // covers, enumerated pair-major into 32-slot groups
    {
        SlotBox& b = ctx->box;
        b.n_pairs = P;
        b.k0 = (int32_t)(first / P);
        b.nk = (int32_t)((end - 1) / P) - b.k0 + 1;
        const int64_t ja = first % P, jb = (end - 1) % P;
        if (ctx->pair_mode) {                            // every operating point of a pair range
            b.j0 = ctx->pair_first;
            b.nj = ctx->pair_count;
        } else if (b.nk == 1) {
            b.j0 = ja;
            b.nj = jb - ja + 1;
        } else if (b.nk == 2 && jb + 1 < ja) {           // two partial rows: pairs ja .. P-1, 0 .. jb
            b.j0 = ja;
            b.nj = P - ja + jb + 1;
        } else {
            b.j0 = 0;
            b.nj = P;
        }
        b.slot_first = first;
        b.slot_end = end;
        ctx->n_grp = (b.nj * b.nk + 31) / 32;
    }
    const int64_t sw_lo = 0, sw_hi = ctx->n_grp;
    const int32_t S = ctx->n_pi + ctx->n_gates;
    std::memset(&ctx->stats, 0, sizeof ctx->stats);

    CK(ctx->d_p1t.ensure((size_t)std::max(ctx->n_pi, 1) * n_pw * 4));
    CK(ctx->d_p2t.ensure((size_t)std::max(ctx->n_pi, 1) * n_pw * 4));
    CK(ctx->d_p1g.ensure((size_t)std::max(ctx->n_pi, 1) * ctx->n_grp * (AVFS_PI_GMAJOR ? 8 : 4)));
    CK(ctx->d_p2g.ensure((size_t)std::max(ctx->n_pi, 1) * ctx->n_grp * 4));
    CK(ctx->d_act.ensure((size_t)S * V * sizeof(unsigned long long)));
    CK(ctx->d_latest.ensure((size_t)V * 4));
    CK(ctx->d_err.ensure(16));
    CK(ctx->d_count.ensure(16));
    CK(cudaMemsetAsync(ctx->d_act.p, 0, (size_t)S * V * sizeof(unsigned long long), ctx->stream));
    CK(cudaMemsetAsync(ctx->d_latest.p, 0, (size_t)V * 4, ctx->stream));
    CK(cudaMemsetAsync(ctx->d_err.p, 0, 16, ctx->stream));
    CK(ctx->d_enc.ensure(8));
    CK(cudaMemsetAsync(ctx->d_enc.p, 0, 8, ctx->stream));
    // delay computation kernel: d'(gate, pin, pol, Vdd) in FP64 ->
    // binary32 table, or (delay_in_sweep) only the d' > 0 check, the sweep
    // then evaluating Eq. (4)/(9) itself for the gates that need delays
    const bool in_sweep = ctx->opt.delay_in_sweep != 0;
    if (!in_sweep) CK(ctx->d_dtab.ensure((size_t)ctx->box.nk * std::max(ctx->n_gates, 1) * 8 * sizeof(float)));
    else ctx->d_dtab.release();
    {
        DelayParams& dp = ctx->dparams;
        dp = DelayParams{};
        dp.dd = ctx->d_ddesc.as<DelayDesc>();
        dp.n_gates = ctx->n_gates;
        dp.coef = ctx->d_coef.as<double>();
        dp.deg_v = ctx->deg_v;
        dp.deg_c = ctx->deg_c;
        dp.vdd = ctx->d_vdd.as<double>();
        dp.n_vdd = V;
        dp.kv_lo = ctx->box.k0;
        dp.kv_hi = ctx->box.k0 + ctx->box.nk;
        dp.n_isl = ctx->n_isl;
        dp.v_min = ctx->v_min;
        dp.v_max = ctx->v_max;
        dp.quantum = ctx->opt.quantum_ps;
        dp.dtab = in_sweep ? nullptr : ctx->d_dtab.as<float>();
        dp.err = ctx->d_err.as<int32_t>();
        CK(launch_delays(dp, ctx->stream));
        ctx->stats.launches++;
    }
    // H4: stimulus expansion (transpose to PI-major 32-pair words)
    CK(launch_expand(ctx->d_p1.as<uint32_t>(), ctx->d_p2.as<uint32_t>(), P, ctx->words, ctx->n_pi, n_pw,
                     ctx->d_p1t.as<uint32_t>(), ctx->d_p2t.as<uint32_t>(), ctx->stream));
    CK(launch_expand_groups(ctx->d_p1.as<uint32_t>(), ctx->d_p2.as<uint32_t>(), ctx->words, ctx->n_pi, ctx->box,
                            ctx->n_grp, ctx->d_p1g.as<uint32_t>(), ctx->d_p2g.as<uint32_t>(), ctx->stream));
    CK(launch_pi_activity(ctx->d_p1t.as<uint32_t>(), ctx->d_p2t.as<uint32_t>(), ctx->n_pi, n_pw, ctx->box, V,
                          ctx->d_act.as<unsigned long long>(), ctx->stream));
    ctx->stats.launches += 3;

    ctx->rounds.clear();
    // rerun rounds' arenas and heaps of the previous simulate are kept for
    // the next one (repeated runs rerun the same groups without reallocating
    // inside the step); pass 0 takes their memory back if it needs it
    // slot batching: when the arena for every slot group would not
    // fit, the groups run in batches on the same arena and heap; activity,
    // latest arrival and energy accumulate over all batches, waveform readback
    // keeps the last batch
    const int64_t n_sw_all = sw_hi - sw_lo;
    const int64_t region0 = region_size(32 * ctx->opt.capacity);
    const int64_t per_group = ((int64_t)ctx->n_pinned + ctx->n_scratch) * (region0 + (int64_t)sizeof(uint4));
    // device bytes one group needs: its arena share plus its expected spill
    // (learned from earlier batches / simulates, words per group)
    auto group_bytes = [&]() { return (double)per_group + 1.25 * 4.0 * (double)ctx->spill_per_group; };
    auto avail_bytes = [&]() -> double {
        size_t fr = 0, tot = 0;
        if (cudaMemGetInfo(&fr, &tot) != cudaSuccess) return 0.0;
        double own = 0;
        for (auto& a : ctx->arena) own += (double)a.n;
        for (auto& a : ctx->recs) own += (double)a.n;
        for (auto& h : ctx->spill) own += (double)h.n;
        return (double)fr + own - (double)(2ll << 30);
    };
    int64_t nb = n_sw_all;
    bool learn = false;                                 // first batch only one wave: learn the spill per group
    if (ctx->opt.max_batch_slots > 0) {
        nb = std::max<int64_t>(1, ctx->opt.max_batch_slots / 32);
    } else if (!ctx->arena.empty() && !ctx->recs.empty() &&
               ctx->arena[0].n >= (size_t)(n_sw_all * ((int64_t)ctx->n_pinned + ctx->n_scratch) * region0) &&
               ctx->recs[0].n >= (size_t)(n_sw_all * ((int64_t)ctx->n_pinned + ctx->n_scratch) * (int64_t)sizeof(uint4)) &&
               ctx->spill_per_group * n_sw_all * 5 / 4 <= (int64_t)(ctx->spill.empty() ? 0 : ctx->spill[0].n / 4)) {
        // fits the arena, records and heap of a previous simulate: no device
        // memory query (cudaMemGetInfo costs milliseconds at times)
        nb = n_sw_all;
    } else {
        const double av = avail_bytes();
        const int64_t fit = (int64_t)(0.8 * av / std::max(group_bytes(), 1.0));
        if (fit < n_sw_all) {
            nb = std::max<int64_t>(1, fit);
            if (!ctx->spill_known) { nb = std::min<int64_t>(nb, (int64_t)ctx->n_sm); learn = true; }
        } else if (!ctx->spill_known && (double)per_group * (double)n_sw_all > 0.5 * av && n_sw_all > ctx->n_sm) {
            // the arena alone would take most of the memory and the spill of
            // this netlist is not known yet: learn it on one wave first
            nb = (int64_t)ctx->n_sm;
            learn = true;
        }
    }
    nb = std::min(nb, n_sw_all);
    ctx->n_batches = 0;
    ctx->pend_sweep_ms = 0;
    ctx->pend_hint = 0;
    for (int64_t b0 = sw_lo; b0 < sw_hi; b0 += nb) {
    if (b0 > sw_lo) {                                   // earlier batches' rerun memory is not kept
        for (size_t r = 1; r < ctx->arena.size(); ++r) ctx->arena[r].release();
        for (size_t r = 1; r < ctx->recs.size(); ++r) ctx->recs[r].release();
        for (size_t r = 1; r < ctx->spill.size(); ++r) ctx->spill[r].release();
        if (learn && ctx->opt.max_batch_slots <= 0) {   // resize the remaining batches
            const int64_t fit = (int64_t)(0.8 * avail_bytes() / std::max(group_bytes(), 1.0));
            nb = std::max<int64_t>(1, std::min(fit, sw_hi - b0));
            learn = false;
        }
    }
    ctx->n_batches++;
    ctx->rounds.clear();
    Round R0;
    const bool learning = learn && b0 == sw_lo;
    R0.n_sw = std::min(nb, sw_hi - b0);
    R0.sw_first = b0;
    R0.capacity = ctx->opt.capacity;
    R0.W = 32 * R0.capacity;
    R0.region_bytes = region_size(R0.W);
    {
        const int64_t arena_words = ((int64_t)ctx->n_pinned + ctx->n_scratch) * R0.n_sw * R0.region_bytes / 4;
        // auto: arena/4 (>= 256 MiB), or 1.25x what the previous simulate asked
        // for in all its rounds, so that repeated runs do not rerun
        R0.spill_want = ctx->opt.spill_bytes > 0 ? ctx->opt.spill_bytes / 4
                      : ctx->opt.spill_bytes < 0 ? 0
                      : std::max<int64_t>({arena_words / 4, (256ll << 20) / 4,
                                           ctx->spill_per_group * R0.n_sw + ctx->spill_per_group * R0.n_sw / 4});
        R0.spill_exact = ctx->opt.spill_bytes > 0;
        // the first batch of a run that must learn the spill per group (one
        // wave): give its heap most of the free memory rather than a guess
        if (learning && ctx->opt.spill_bytes == 0)
            R0.spill_want = std::max<int64_t>(R0.spill_want, (int64_t)(0.6 * avail_bytes() / 4.0 / 1.25));
    }
    if (getenv("AVFS_DEBUG"))
        fprintf(stderr, "[avfs] batch %d: groups [%lld, %lld) of %lld, heap want %.2f GB%s\n", ctx->n_batches,
                (long long)b0, (long long)(b0 + R0.n_sw), (long long)n_sw_all, 4e-9 * (double)R0.spill_want,
                learning ? " (learning)" : "");
    st = run_round(ctx, R0, 0, nullptr, nullptr, ctx->opt.profile != 0);
    if (st != AVFS_OK) return st;
    ctx->rounds.push_back(R0);
    st = issue_checks(ctx, 0, 0);
    if (st != AVFS_OK) return st;
    ctx->pend_r = 0;
    ctx->pend_cur = 0;
    ctx->pend_r0n = std::max<int64_t>(R0.n_sw, 1);
    if (b0 + nb < sw_hi) {                              // more batches follow: settle this one now
        st = settle_batch(ctx);
        if (st != AVFS_OK) return st;
    }
    }  // batches
    ctx->pend_t0 = t0;
    const int64_t n_sim = ctx->pair_mode ? ctx->box.nj * ctx->box.nk : end - first;
    ctx->pend_slots = n_sim;
    ctx->stats.slots = n_sim;
    ctx->stats.evals = (int64_t)ctx->n_gates * n_sim;
    ctx->stats.slot_warps = sw_hi - sw_lo;
    ctx->stats.grid = ctx->rounds[0].grid;
    ctx->stats.n_scratch_buffers = ctx->n_scratch;
    ctx->stats.n_pinned = ctx->n_pinned;
    ctx->pending = true;                               // the last batch's overflow check is outstanding
    return AVFS_OK;
}

avfs_status avfs_get_activity(avfs_ctx* ctx, uint64_t* out, int32_t out_is_device) {
    CHECK_CTX();
    SETTLE();
    if (!out) return fail(ctx, AVFS_ERR_ARG, "null output");
    if (!ctx->sim_done) return fail(ctx, AVFS_ERR_STATE, "simulate first");
    const size_t n = (size_t)(ctx->n_pi + ctx->n_gates) * ctx->vdd.size() * sizeof(uint64_t);
    CK(cudaMemcpyAsync(out, ctx->d_act.p, n, out_is_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost,
                       ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    return AVFS_OK;
}

avfs_status avfs_get_latest_arrival(avfs_ctx* ctx, float* out, int32_t out_is_device) {
    CHECK_CTX();
    SETTLE();
    if (!out) return fail(ctx, AVFS_ERR_ARG, "null output");
    if (!ctx->sim_done) return fail(ctx, AVFS_ERR_STATE, "simulate first");
    CK(cudaMemcpyAsync(out, ctx->d_latest.p, ctx->vdd.size() * 4,
                       out_is_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, ctx->stream));
    if (!out_is_device) CK(cudaStreamSynchronize(ctx->stream));
    return AVFS_OK;
}

// device map slot group -> (round holding its final data, index in that round)
static avfs_status ensure_round_map(avfs_ctx* ctx) {
    const int64_t n_sw_total = std::max<int64_t>(ctx->n_grp, 1);
    if (!ctx->map_valid) {
        std::vector<int32_t> rnd(n_sw_total, -1), idx(n_sw_total, 0);
        for (size_t r = 0; r < ctx->rounds.size(); ++r) {
            const Round& R = ctx->rounds[r];
            for (int64_t i = 0; i < R.n_sw; ++i) {
                const int64_t sw = R.sws.empty() ? R.sw_first + i : R.sws[i];
                rnd[sw] = (int32_t)r;
                idx[sw] = (int32_t)i;
            }
        }
        CK(ctx->d_swround.ensure(n_sw_total * 4));
        CK(ctx->d_swindex.ensure(n_sw_total * 4));
        CK(cudaMemcpy(ctx->d_swround.p, rnd.data(), n_sw_total * 4, cudaMemcpyHostToDevice));
        CK(cudaMemcpy(ctx->d_swindex.p, idx.data(), n_sw_total * 4, cudaMemcpyHostToDevice));
        ctx->map_valid = true;
    }
    return AVFS_OK;
}

static avfs_status gather(avfs_ctx* ctx, int32_t n_sig, const int32_t* sig, int64_t slot0, int64_t n_slots,
                          int32_t cap, uint8_t* init, int32_t* count, float* times) {
    if (!ctx->sim_done) return fail(ctx, AVFS_ERR_STATE, "simulate first");
    if (n_sig < 0 || n_slots < 0 || cap < 0 || (n_sig > 0 && !sig)) return fail(ctx, AVFS_ERR_ARG, "bad readback arguments");
    if (slot0 < ctx->sim_first || slot0 + n_slots > ctx->sim_end)
        return fail(ctx, AVFS_ERR_ARG, "slots [%lld, %lld) outside the simulated range [%lld, %lld)",
                    (long long)slot0, (long long)(slot0 + n_slots), (long long)ctx->sim_first, (long long)ctx->sim_end);
    if (ctx->pair_mode)
        for (int64_t s = slot0; s < slot0 + n_slots; ++s)
            if ((s % ctx->n_pairs) - ctx->pair_first < 0 || (s % ctx->n_pairs) - ctx->pair_first >= ctx->pair_count)
                return fail(ctx, AVFS_ERR_ARG, "slot %lld (pair %lld) outside the simulated pair range [%lld, %lld)",
                            (long long)s, (long long)(s % ctx->n_pairs), (long long)ctx->pair_first,
                            (long long)(ctx->pair_first + ctx->pair_count));
    if (ctx->rounds.size() > 8) return fail(ctx, AVFS_ERR_STATE, "too many rounds");
    std::vector<uint32_t> sl(n_sig);
    for (int32_t i = 0; i < n_sig; ++i) {
        if (sig[i] < 0 || sig[i] >= ctx->n_pi + ctx->n_gates) return fail(ctx, AVFS_ERR_ARG, "signal %d out of range", sig[i]);
        sl[i] = ctx->loc[sig[i]];
        if ((sl[i] & LOC_KIND) == LOC_SCRATCH)
            return fail(ctx, AVFS_ERR_ARG, "signal %d is not kept (not a PO/probe; use keep_all)", sig[i]);
        if ((sl[i] & LOC_KIND) == LOC_PINNED) sl[i] = LOC_PINNED | buffer_id(ctx, sl[i]);
    }
    if (n_sig == 0 || n_slots == 0) return AVFS_OK;
    const int32_t n_pw = (int32_t)((ctx->n_pairs + 31) / 32);
    {
        avfs_status ms = ensure_round_map(ctx);
        if (ms != AVFS_OK) return ms;
    }
    const size_t n = (size_t)n_sig * n_slots;
    CK(ctx->g_loc.ensure(n_sig * 4));
    CK(ctx->g_init.ensure(n));
    CK(ctx->g_count.ensure(n * 4));
    if (times) CK(ctx->g_times.ensure(std::max<size_t>(n * cap * 4, 4)));
    CK(ctx->g_bad.ensure(4));
    CK(cudaMemcpy(ctx->g_loc.p, sl.data(), n_sig * 4, cudaMemcpyHostToDevice));
    CK(cudaMemsetAsync(ctx->g_bad.p, 0, 4, ctx->stream));
    GatherParams g{};
    g.sig_loc = ctx->g_loc.as<uint32_t>();
    g.n_sig = n_sig;
    g.slot0 = slot0;
    g.n_slots = n_slots;
    g.box = ctx->box;
    g.n_pw = n_pw;
    g.p1t = ctx->d_p1t.as<uint32_t>();
    g.p2t = ctx->d_p2t.as<uint32_t>();
    g.sw_round = ctx->d_swround.as<int32_t>();
    g.sw_index = ctx->d_swindex.as<int32_t>();
    for (size_t r = 0; r < ctx->rounds.size(); ++r)
        g.rounds[r] = GatherRound{ctx->arena[r].as<uint8_t>(), ctx->recs[r].as<uint4>(), ctx->rounds[r].region_bytes,
                                  ctx->rounds[r].n_sw, (int64_t)ctx->n_pinned + ctx->n_scratch};
    g.cap = times ? cap : 0;
    g.init = ctx->g_init.as<uint8_t>();
    g.count = ctx->g_count.as<int32_t>();
    g.times = times ? ctx->g_times.as<float>() : nullptr;
    g.bad = ctx->g_bad.as<int32_t>();
    CK(launch_gather(g, ctx->stream));
    int32_t bad = 0;
    CK(cudaMemcpyAsync(&bad, ctx->g_bad.p, 4, cudaMemcpyDeviceToHost, ctx->stream));
    if (init) CK(cudaMemcpyAsync(init, ctx->g_init.p, n, cudaMemcpyDeviceToHost, ctx->stream));
    if (count) CK(cudaMemcpyAsync(count, ctx->g_count.p, n * 4, cudaMemcpyDeviceToHost, ctx->stream));
    if (times && cap > 0) CK(cudaMemcpyAsync(times, ctx->g_times.p, n * cap * 4, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    if (bad && ctx->n_batches > 1)
        return fail(ctx, AVFS_ERR_STATE, "waveforms of slots outside the last of %d batches are not retained "
                    "(raise max_batch_slots or restrict the slot range)", ctx->n_batches);
    if (bad) return fail(ctx, AVFS_ERR_STATE, "readback hit slots without valid data (code %d)", bad);
    return AVFS_OK;
}

avfs_status avfs_get_final_values(avfs_ctx* ctx, int32_t n_sig, const int32_t* sig, int64_t slot0,
                                  int64_t n_slots, uint8_t* out) {
    CHECK_CTX();
    SETTLE();
    if (!out) return fail(ctx, AVFS_ERR_ARG, "null output");
    const size_t n = (size_t)std::max(n_sig, 0) * std::max<int64_t>(n_slots, 0);
    std::vector<uint8_t> init(n);
    std::vector<int32_t> cnt(n);
    avfs_status st = gather(ctx, n_sig, sig, slot0, n_slots, 0, init.data(), cnt.data(), nullptr);
    if (st != AVFS_OK) return st;
    for (size_t i = 0; i < n; ++i) out[i] = (uint8_t)(init[i] ^ (cnt[i] & 1));
    return AVFS_OK;
}

avfs_status avfs_get_waveforms(avfs_ctx* ctx, int32_t n_sig, const int32_t* sig, int64_t slot0, int64_t n_slots,
                               int32_t cap, uint8_t* init, int32_t* count, float* times) {
    CHECK_CTX();
    SETTLE();
    if (!init || !count || (cap > 0 && !times)) return fail(ctx, AVFS_ERR_ARG, "null output");
    return gather(ctx, n_sig, sig, slot0, n_slots, cap, init, count, cap > 0 ? times : nullptr);
}

avfs_status avfs_capture(avfs_ctx* ctx, const float* t_clk, int32_t n_bins, float lo_ps, float width_ps,
                         uint32_t* fail_pairs, uint32_t* fail_po, uint32_t* slack_hist, uint8_t* fail_bits) {
    CHECK_CTX();
    SETTLE();
    if (!ctx->sim_done) return fail(ctx, AVFS_ERR_STATE, "simulate first");
    if (!t_clk || !fail_pairs) return fail(ctx, AVFS_ERR_ARG, "null t_clk / fail_pairs");
    if (slack_hist && (n_bins < 1 || !(width_ps > 0))) return fail(ctx, AVFS_ERR_ARG, "bad histogram bins");
    if (ctx->rounds.size() > 8) return fail(ctx, AVFS_ERR_STATE, "too many rounds");
    if (ctx->n_batches > 1)
        return fail(ctx, AVFS_ERR_STATE, "capture needs every slot's PO waveforms; the last simulate ran in %d batches "
                    "(raise max_batch_slots or restrict the slot range)", ctx->n_batches);
    avfs_status ms = ensure_round_map(ctx);
    if (ms != AVFS_OK) return ms;
    const int32_t V = (int32_t)ctx->vdd.size();
    const int32_t n_po = (int32_t)ctx->po.size();
    const int32_t n_pw = (int32_t)((ctx->n_pairs + 31) / 32);
    const Round& R0 = ctx->rounds[0];
    const int64_t n_sw = R0.n_sw, n_slots = ctx->pair_mode ? ctx->box.nj * ctx->box.nk : ctx->sim_end - ctx->sim_first;
    std::vector<uint32_t> loc(std::max(n_po, 1));
    for (int32_t o = 0; o < n_po; ++o) {
        const uint32_t l = ctx->loc[ctx->po[o]];
        loc[o] = (l & LOC_KIND) == LOC_PI ? l : (LOC_PINNED | buffer_id(ctx, l));
    }
    const size_t nb = slack_hist ? (size_t)n_bins : 0;
    // device scratch: loc | t_clk | slot_fail, slot_last | fail_po, fail_pairs, hist | fail_bits
    CK(ctx->c_loc.ensure(loc.size() * 4));
    CK(ctx->c_tclk.ensure((size_t)V * 4));
    CK(ctx->c_slot.ensure((size_t)n_sw * 32 * 8));
    const size_t out_words = (size_t)n_po * V + V + (size_t)V * nb;
    CK(ctx->c_out.ensure(out_words * 4 + (size_t)n_slots + 16));
    CK(cudaMemcpy(ctx->c_loc.p, loc.data(), loc.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(ctx->c_tclk.p, t_clk, (size_t)V * 4, cudaMemcpyHostToDevice));
    CK(cudaMemsetAsync(ctx->c_slot.p, 0, (size_t)n_sw * 32 * 8, ctx->stream));
    CK(cudaMemsetAsync(ctx->c_out.p, 0, out_words * 4, ctx->stream));
    CaptureParams p{};
    p.po_loc = ctx->c_loc.as<uint32_t>();
    p.n_po = n_po;
    p.n_vdd = V;
    p.t_clk = ctx->c_tclk.as<float>();
    p.sw_lo = R0.sw_first;
    p.n_sw = n_sw;
    p.box = ctx->box;
    p.n_pw = n_pw;
    p.p1t = ctx->d_p1t.as<uint32_t>();
    p.p2t = ctx->d_p2t.as<uint32_t>();
    p.sw_round = ctx->d_swround.as<int32_t>();
    p.sw_index = ctx->d_swindex.as<int32_t>();
    for (size_t r = 0; r < ctx->rounds.size(); ++r)
        p.rounds[r] = GatherRound{ctx->arena[r].as<uint8_t>(), ctx->recs[r].as<uint4>(), ctx->rounds[r].region_bytes,
                                  ctx->rounds[r].n_sw, (int64_t)ctx->n_pinned + ctx->n_scratch};
    p.slot_fail = ctx->c_slot.as<uint32_t>();
    p.slot_last = ctx->c_slot.as<uint32_t>() + (size_t)n_sw * 32;
    p.fail_po = ctx->c_out.as<uint32_t>();
    p.fail_pairs = p.fail_po + (size_t)n_po * V;
    p.hist = slack_hist ? p.fail_pairs + V : nullptr;
    p.n_bins = std::max(n_bins, 1);
    p.lo = lo_ps;
    p.width = width_ps > 0 ? width_ps : 1.0f;
    p.fb_pairs = ctx->pair_mode ? 1 : 0;
    p.fail_bits = fail_bits ? reinterpret_cast<uint8_t*>(p.fail_pairs + V + (size_t)V * nb) : nullptr;
    CK(launch_capture(p, ctx->stream));
    CK(cudaMemcpyAsync(fail_pairs, p.fail_pairs, (size_t)V * 4, cudaMemcpyDeviceToHost, ctx->stream));
    if (fail_po && n_po) CK(cudaMemcpyAsync(fail_po, p.fail_po, (size_t)n_po * V * 4, cudaMemcpyDeviceToHost, ctx->stream));
    if (slack_hist) CK(cudaMemcpyAsync(slack_hist, p.hist, (size_t)V * nb * 4, cudaMemcpyDeviceToHost, ctx->stream));
    if (fail_bits) CK(cudaMemcpyAsync(fail_bits, p.fail_bits, (size_t)n_slots, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    return AVFS_OK;
}

avfs_status avfs_get_switching_energy(avfs_ctx* ctx, double* out) {
    CHECK_CTX();
    SETTLE();
    if (!out) return fail(ctx, AVFS_ERR_ARG, "null output");
    if (!ctx->sim_done) return fail(ctx, AVFS_ERR_STATE, "simulate first");
    const int32_t V = (int32_t)ctx->vdd.size();
    CK(ctx->d_energy.ensure((size_t)V * sizeof(double)));
    CK(cudaMemsetAsync(ctx->d_energy.p, 0, (size_t)V * sizeof(double), ctx->stream));
    CK(launch_energy(ctx->d_act.as<unsigned long long>(), ctx->d_cload.as<double>(), ctx->d_vdd.as<double>(),
                     ctx->d_island.as<int32_t>(), ctx->n_isl, ctx->n_pi, ctx->n_gates, V, ctx->d_energy.as<double>(),
                     ctx->stream));
    CK(cudaMemcpyAsync(out, ctx->d_energy.p, (size_t)V * sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    return AVFS_OK;
}

avfs_status avfs_get_timing(avfs_ctx* ctx, double* sweep_ms, double* rerun_ms) {
    CHECK_CTX();
    SETTLE();
    if (!sweep_ms || !rerun_ms) return fail(ctx, AVFS_ERR_ARG, "null output");
    if (!ctx->sim_done) return fail(ctx, AVFS_ERR_STATE, "simulate first");
    *sweep_ms = ctx->stats.sweep_ms;
    *rerun_ms = ctx->stats.rerun_ms;
    return AVFS_OK;
}

int32_t avfs_debug_phase_cycles(uint64_t* out16, int32_t reset) {
    return debug_phase_cycles(reinterpret_cast<unsigned long long*>(out16), reset);
}

avfs_status avfs_get_stats(avfs_ctx* ctx, avfs_stats* st) {
    CHECK_CTX();
    SETTLE();
    if (!st) return fail(ctx, AVFS_ERR_ARG, "null output");
    if (!ctx->sim_done) return fail(ctx, AVFS_ERR_STATE, "simulate first");
    // algorithmic bytes of the sweep: every signal's
    // waveform (PIs included) is written once and read once per reading pin,
    // 4 B header per slot plus 4 B per transition.
    const int32_t V = (int32_t)ctx->vdd.size();
    const int32_t S = ctx->n_pi + ctx->n_gates;
    std::vector<uint64_t> act((size_t)S * V);
    CK(cudaMemcpy(act.data(), ctx->d_act.p, act.size() * 8, cudaMemcpyDeviceToHost));
    const double slots = (double)ctx->stats.slots;
    double b = 0;
    for (int32_t s = 0; s < S; ++s) {
        uint64_t a = 0;
        for (int32_t k = 0; k < V; ++k) a += act[(size_t)s * V + k];
        b += (1.0 + (double)ctx->fanout[s]) * (4.0 * slots + 4.0 * (double)a);
    }
    ctx->stats.alg_bytes = (int64_t)b;
    // the same for the encoding the sweep moves: per (gate
    // output, slot group) a 16-B record, per slot with events a 4-B entry,
    // 4 B per transition, each written once and read once per reading pin;
    // PI waveforms are the stimulus words (8 B per (PI, group) per reading pin)
    unsigned long long units = 0;
    CK(cudaMemcpy(&units, ctx->d_enc.p, 8, cudaMemcpyDeviceToHost));
    const double groups = (double)ctx->stats.slot_warps;
    double e = 4.0 * (double)units;
    for (int32_t s = 0; s < S; ++s) {
        uint64_t a = 0;
        for (int32_t k = 0; k < V; ++k) a += act[(size_t)s * V + k];
        if (s < ctx->n_pi) e += (double)ctx->fanout[s] * 8.0 * groups;
        else e += (1.0 + (double)ctx->fanout[s]) * (16.0 * groups + 4.0 * (double)a);
    }
    ctx->stats.enc_bytes = (int64_t)e;
    *st = ctx->stats;
    return AVFS_OK;
}

}  // extern "C"
