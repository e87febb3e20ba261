// avfs_kernels.cu -- sm_100a kernels of the AVFS time-simulation hot path.
//
// Paper: Schneider & Wunderlich, DATE'20 (/root/reference/PAPER.md, "P:L<n>").
//
//   expand_kernel       H4  stimulus expansion: pair-major packed bits ->
//                           PI-major bit-transposed words, one u32 per
//                           (PI, 32-pair group), so a warp of 32 slots reads
//                           its PI waveforms with one broadcast load
//                           (P:L141 step 3).
//   pi_activity_kernel  H8  PI switching activity per operating point.
//   sweep_kernel        H6+H7 persistent level sweep.  One CTA owns one
//                           32-slot group (same Vdd, 32 stimulus pairs) at a
//                           time and walks every level of the netlist with a
//                           CTA barrier between levels (P:L166 level-wise
//                           processing); warp w evaluates gates w, w+nw, ...
//                           of the level for the 32 slots (the
//                           horizontal plane = one gate, all slots).  Per
//                           gate: FP64 Horner delays lane-parallel (P:L139,
//                           P:L152-L160 steps 1-5, Eq. 9), coalesced header
//                           loads, cp.async 16-B staging of the compact input
//                           event lists into shared memory, per-slot k-way
//                           merge with the inertial filter (reading
//                           C3-C6), compaction of the outputs through shared
//                           memory, 128-bit stores, warp-ballot overflow
//                           detection and activity / latest-arrival
//                           reductions (P:L141 step 4).
//   compact_kernel      H7  list of overflowed slot groups for the rerun.
//   gather_kernel       H9  readback of kept waveforms.
#include <cuda_runtime.h>
#include <cstdint>

#include "avfs_internal.h"

namespace avfs {

// Waveforms are produced and consumed inside one launch: read them at L2
// (.cg), never through a possibly stale L1 line.
__device__ __forceinline__ uint32_t ld_u32(const void* p) {
    return __ldcg(reinterpret_cast<const unsigned int*>(p));
}

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
    uint32_t s = static_cast<uint32_t>(__cvta_generic_to_shared(smem));
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async16_a(uint32_t s, const void* gmem) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem) : "memory");
}
// TMA bulk copy global -> shared, completion signalled on an mbarrier (tx bytes)
__device__ __forceinline__ void tma_bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n"
                 ::"r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_init(uint32_t bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(bar) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t phase) {
    asm volatile(
        "{\n .reg .pred P;\n WAIT_%=:\n"
        " mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n"
        " @!P bra WAIT_%=;\n}\n" ::"r"(bar), "r"(phase) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_global() {
    asm volatile("fence.proxy.async.global;\n" ::: "memory");
}
__device__ __forceinline__ void cp_async_wait_all() {
    asm volatile("cp.async.wait_all;\n" ::: "memory");
}
__device__ __forceinline__ void st_global_v4(void* p, float4 v) {
    asm volatile("st.global.v4.f32 [%0], {%1, %2, %3, %4};\n" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z),
                 "f"(v.w)
                 : "memory");
}

__device__ __forceinline__ uint32_t warp_incl_scan(uint32_t v, int lane) {
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t u = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += u;
    }
    return v;
}

// ---------------------------------------------------------------------------
// Delay computation kernel (P:L139, P:L152-L160 steps 3-5): one thread per
// (operating point, gate, pin, polarity).  f(P) of Eq. (4) by Horner with FMA
// in FP64, d' = d_nom (1 + f) (Eq. 9), optional Q-mode rounding
// (reading C12), rounded once to binary32 (reading C11).  The sweep reads the
// 8 delays of a gate as two uniform float4 loads per 32 slots.
// ---------------------------------------------------------------------------
__global__ void delay_kernel(const DelayParams p) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t total = (int64_t)p.n_vdd * p.n_gates * 8;
    if (t >= total) return;
    const int e = (int)(t & 7);
    const int64_t vg = t >> 3;
    const int g = (int)(vg % p.n_gates);
    const int kv = (int)(vg / p.n_gates);
    const DelayDesc& D = p.dd[g];
    float out = 1.0f;
    if (e < 2 * (int)D.k) {
        const double v = p.vdd[(size_t)kv * p.n_isl + D.island];           // gate's island supply (NEXT-2)
        const double x = (v - p.v_min) / (p.v_max - p.v_min);                // phi_V
        const double* cf = p.coef + D.coef_off + e * (p.deg_v + 1);
        double f = cf[p.deg_v];
        for (int i = p.deg_v - 1; i >= 0; --i) f = fma(f, x, cf[i]);
        double d = D.dnom[e] * (1.0 + f);
        if (p.quantum > 0.0) d = p.quantum * rint(d / p.quantum);
        if (!(d > 0.0)) atomicOr(p.err, 1);
        out = __double2float_rn(d);
    }
    p.dtab[t] = out;
}

cudaError_t launch_delays(const DelayParams& p, cudaStream_t st) {
    const int64_t n = (int64_t)p.n_vdd * p.n_gates * 8;
    if (n == 0) return cudaSuccess;
    delay_kernel<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(p);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// Per-slot merge of the K sorted input event lists of a gate with the inertial
// filter (reading C3: the pending last output event is cancelled iff
// it lies strictly after the input event; C4: no reschedule on confirming
// events; C5: ties in time are taken in ascending pin order).  Branch-free
// bodies; the element after each head is prefetched from shared memory one
// step ahead.  Returns the exact output count; the first `cstage` surviving
// events are left in shared memory rows s_out[i][lane].
// ---------------------------------------------------------------------------
__device__ __forceinline__ float lds_f32(uint32_t addr) {
    float v;
    asm volatile("ld.shared.f32 %0, [%1];\n" : "=f"(v) : "r"(addr));
    return v;
}
__device__ __forceinline__ void sts_f32(uint32_t addr, float v) {
    asm volatile("st.shared.f32 [%0], %1;\n" ::"r"(addr), "f"(v) : "memory");
}

#define AVFS_INF __int_as_float(0x7f800000)

// filter step shared by all merges: one input event at time t whose pin flip
// gives evaluated output y; d_r / d_f = the pin's rise / fall delays.
struct OutState {
    int n;          // surviving output events
    float tl;       // time of the last surviving event (-inf if it is <= every later input)
    uint32_t proj;  // projected output value
};

__device__ __forceinline__ void filter_step(OutState& o, float t, uint32_t y, float d_r, float d_f,
                                            uint32_t s_out_lane, int cstage) {
    const bool change = y != o.proj;
    const bool cancel = change && (o.tl > t);   // pending output lies after t: pulse filtered
    const bool push = change && !cancel;
    const float tn = t + (y ? d_r : d_f);
    // unconditional store to the next free row (clamped): harmless unless pushed
    sts_f32(s_out_lane + 128u * (uint32_t)min(o.n, cstage), tn);
    o.n += push ? 1 : (cancel ? -1 : 0);
    o.tl = push ? tn : (cancel ? -AVFS_INF : o.tl);   // after a cancel the last event is <= t
    o.proj = y;
}

// one input (BUF / INV / any 1-input cell)
__device__ __forceinline__ int merge1(uint32_t s_in, int c, int n, float d_f, float d_r, uint32_t tt,
                                     uint32_t bits, uint32_t proj, uint32_t s_out_lane, int cstage) {
    const int e = c + n;
    const float a0 = lds_f32(s_in + 4u * (uint32_t)c);
    const float a1 = lds_f32(s_in + 4u * (uint32_t)(c + 1));
    float h = n > 0 ? a0 : AVFS_INF;
    float nh = n > 1 ? a1 : AVFS_INF;
    OutState o{0, -AVFS_INF, proj};
    while (h < AVFS_INF) {
        const float t = h;
        ++c;
        const float raw = lds_f32(s_in + 4u * (uint32_t)(c + 1));
        h = nh;
        nh = (c + 1 < e) ? raw : AVFS_INF;
        bits ^= 1u;
        filter_step(o, t, (tt >> bits) & 1u, d_r, d_f, s_out_lane, cstage);
    }
    return o.n;
}

// two inputs, hand-specialised (62 % of gates on the random DAGs)
__device__ __forceinline__ int merge2(uint32_t s_in, int c0, int n0, int c1, int n1,
                                     const float (&dl)[8], uint32_t tt, uint32_t bits, uint32_t proj,
                                     uint32_t s_out_lane, int cstage) {
    const int e0 = c0 + n0, e1 = c1 + n1;
    float h0, h1, nh0, nh1;
    {
        const float a = lds_f32(s_in + 4u * (uint32_t)c0), b = lds_f32(s_in + 4u * (uint32_t)(c0 + 1));
        const float x = lds_f32(s_in + 4u * (uint32_t)c1), z = lds_f32(s_in + 4u * (uint32_t)(c1 + 1));
        h0 = n0 > 0 ? a : AVFS_INF;
        nh0 = n0 > 1 ? b : AVFS_INF;
        h1 = n1 > 0 ? x : AVFS_INF;
        nh1 = n1 > 1 ? z : AVFS_INF;
    }
    OutState o{0, -AVFS_INF, proj};
    for (;;) {
        const bool p1 = h1 < h0;                 // ties: pin 0 first
        const float t = p1 ? h1 : h0;
        if (!(t < AVFS_INF)) break;
        const int cn = (p1 ? c1 : c0) + 1;
        const int en = p1 ? e1 : e0;
        const float raw = lds_f32(s_in + 4u * (uint32_t)(cn + 1));
        const float hn = p1 ? nh1 : nh0;
        const float nn = (cn + 1 < en) ? raw : AVFS_INF;
        if (p1) { h1 = hn; nh1 = nn; c1 = cn; } else { h0 = hn; nh0 = nn; c0 = cn; }
        bits ^= p1 ? 2u : 1u;
        filter_step(o, t, (tt >> bits) & 1u, p1 ? dl[3] : dl[1], p1 ? dl[2] : dl[0], s_out_lane, cstage);
    }
    return o.n;
}

// generic K (3 and 4 inputs)
template <int K>
__device__ __forceinline__ int merge_k(uint32_t s_in, const int (&cb)[KMAX], const int (&n)[KMAX],
                                       const float (&dl)[8], uint32_t tt, uint32_t bits,
                                       uint32_t proj, uint32_t s_out_lane, int cstage) {
    float h[K], nh[K];
    int c[K], e[K];
#pragma unroll
    for (int q = 0; q < K; ++q) {
        c[q] = cb[q];
        e[q] = cb[q] + n[q];
        const float a0 = lds_f32(s_in + 4u * (uint32_t)c[q]);
        const float a1 = lds_f32(s_in + 4u * (uint32_t)(c[q] + 1));
        h[q] = n[q] > 0 ? a0 : AVFS_INF;
        nh[q] = n[q] > 1 ? a1 : AVFS_INF;
    }
    OutState o{0, -AVFS_INF, proj};
    for (;;) {
        float t = h[0];
        int pm = 0;
#pragma unroll
        for (int q = 1; q < K; ++q) {
            const bool lt = h[q] < t;
            t = lt ? h[q] : t;
            pm = lt ? q : pm;
        }
        if (!(t < AVFS_INF)) break;
        int cn = c[0], en = e[0];
        float hn = nh[0], dfp = dl[0], drp = dl[1];
#pragma unroll
        for (int q = 1; q < K; ++q)
            if (pm == q) { cn = c[q]; en = e[q]; hn = nh[q]; dfp = dl[2 * q]; drp = dl[2 * q + 1]; }
        ++cn;
        const float raw = lds_f32(s_in + 4u * (uint32_t)(cn + 1));
        const float nn = (cn + 1 < en) ? raw : AVFS_INF;
#pragma unroll
        for (int q = 0; q < K; ++q)
            if (pm == q) { c[q] = cn; h[q] = hn; nh[q] = nn; }
        bits ^= 1u << pm;
        filter_step(o, t, (tt >> bits) & 1u, drp, dfp, s_out_lane, cstage);
    }
    return o.n;
}

// Where one warp's 32 slots live for the gate being evaluated.  All regions
// of a round live in one arena [buffer][slot group][region] (buffers: PIs,
// kept signals, scratch), so a region address is one multiply-add.
struct Env {
    uint8_t* row;                  // arena + i * region_bytes
    uint32_t stride;               // bytes between buffers = n_sw * region_bytes (< 4 GiB, checked on host)
    int64_t i;                     // index of the slot group in the round (overflow flag)
    int kv, lane;
    uint32_t s_in_a;               // per-warp input staging (shared window address)
    uint32_t s_out_a;              // per-warp output rows + 4*lane
    uint32_t bar;                  // per-warp mbarrier for the TMA staging
    uint32_t phase;                // its current parity
    unsigned long long* act_kv;    // &act[0][kv]
};

__device__ __forceinline__ uint8_t* region(uint32_t buf, const Env& E) {
    return E.row + (uint64_t)buf * (uint64_t)E.stride;
}

// One gate for one 32-slot group: input headers,
// compact staging, merge/filter, output compaction, reductions.
template <int K>
__device__ __forceinline__ void eval_gate(const SweepParams& p, Env& E, const uint4 ins, const uint4 hd,
                                          const float (&dl)[8]) {
    const int lane = E.lane;
    const uint32_t out_loc = hd.x, sig = hd.y;
    const uint32_t tt = hd.z & 0xffffu;
    const uint32_t in_loc[KMAX] = {ins.x, ins.y, ins.z, ins.w};
    // all input header loads first (one coalesced 128-B row per input)
    const uint8_t* rg[KMAX];
    uint32_t hw[KMAX];
#pragma unroll
    for (int q = 0; q < K; ++q) {
        rg[q] = region(in_loc[q], E);
        hw[q] = __ldcg(reinterpret_cast<const uint32_t*>(rg[q]) + lane);
    }
    int n[KMAX], cb[KMAX];
    uint32_t bits = 0, pois = 0, prevp = 0;
    int sum = 0;
#pragma unroll
    for (int q = 0; q < KMAX; ++q) {
        n[q] = 0;
        cb[q] = 0;
        if (q < K) {
            const uint32_t h = hw[q];
            n[q] = (int)(h & HDR_N);
            cb[q] = (int)((h >> HDR_OFF_SHIFT) & HDR_OFF);
            bits |= ((h >> HDR_INIT_SHIFT) & 1u) << q;
            pois |= h;
            prevp |= h;
            sum += n[q];
        }
    }
    const uint32_t y0 = (tt >> bits) & 1u;
    uint8_t* ro = region(out_loc, E);
    uint32_t* ro_hdr = reinterpret_cast<uint32_t*>(ro);
    const bool first_pass = (p.prev_W == 0);
    const bool any_prev = first_pass || __any_sync(0xffffffffu, (prevp & HDR_PREV) != 0);
    if (__any_sync(0xffffffffu, (pois & HDR_POISON) != 0)) {   // upstream overflow: nothing valid here
        __stcg(ro_hdr + lane, HDR_POISON | HDR_PREV | (y0 << HDR_INIT_SHIFT));
        return;
    }
    if (!__any_sync(0xffffffffu, sum != 0)) {                   // no input event in any slot: constant output
        __stcg(ro_hdr + lane, (y0 << HDR_INIT_SHIFT) | (any_prev ? HDR_PREV : 0u));
        return;
    }
    // stage each input's compact event list into shared memory with one TMA
    // bulk copy per input (extent = lane 31's offset + count), one mbarrier
    int stage_base = 0;
    {
        int base = 0;
        int ext[KMAX];
#pragma unroll
        for (int q = 0; q < K; ++q) {
            ext[q] = __shfl_sync(0xffffffffu, cb[q] + n[q], 31);
            ext[q] = (ext[q] + 3) & ~3;
            cb[q] += base;
            base += ext[q];
        }
        if (base > p.stage_words) {                    // inputs exceed this capacity's staging: rerun
            __stcg(ro_hdr + lane, HDR_POISON | HDR_PREV | (y0 << HDR_INIT_SHIFT));
            if (lane == 0) p.ovf[p.i_base + E.i] = 1;
            return;
        }
        stage_base = base;
        if (base > 0) {
            if (lane == 0) {
                fence_proxy_async_smem();              // earlier generic reads of the staging area
                mbar_expect_tx(E.bar, 4u * (uint32_t)base);
                uint32_t dst = E.s_in_a;
#pragma unroll
                for (int q = 0; q < K; ++q) {
                    if (ext[q] > 0) tma_bulk_g2s(dst, rg[q] + 128, 4u * (uint32_t)ext[q], E.bar);
                    dst += 4u * (uint32_t)ext[q];
                }
            }
            mbar_wait(E.bar, E.phase);
            E.phase ^= 1u;
        }
    }
    int n_out;
    if (K == 1) {
        n_out = merge1(E.s_in_a, cb[0], n[0], dl[0], dl[1], tt, bits, y0, E.s_out_a, p.cstage);
    } else if (K == 2) {
        n_out = merge2(E.s_in_a, cb[0], n[0], cb[1], n[1], dl, tt, bits, y0, E.s_out_a, p.cstage);
    } else {
        n_out = merge_k<K>(E.s_in_a, cb, n, dl, tt, bits, y0, E.s_out_a, p.cstage);
    }
    // output: scan, overflow ballot, compact stores row by row (warp-uniform loop)
    const uint32_t incl = warp_incl_scan((uint32_t)n_out, lane);
    const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
    const uint32_t excl = incl - (uint32_t)n_out;
    const bool ovf = __any_sync(0xffffffffu, n_out > p.cstage) || total > (uint32_t)p.W;
    bool prev = true;
    if (!first_pass)
        prev = any_prev || stage_base > p.prev_stage_words || __any_sync(0xffffffffu, n_out > p.prev_cstage) ||
               total > (uint32_t)p.prev_W;
    if (!ovf) {
        const int rows = (int)__reduce_max_sync(0xffffffffu, (uint32_t)n_out);
        float* dst = reinterpret_cast<float*>(ro + 128) + excl;
        for (int r = 0; r < rows; ++r) {
            const float v = lds_f32(E.s_out_a + 128u * (uint32_t)r);
            if (r < n_out) __stcg(dst + r, v);
        }
    } else if (lane == 0) {
        p.ovf[p.i_base + E.i] = 1;
    }
    __stcg(ro_hdr + lane, (uint32_t)min(n_out, (int)HDR_N) | ((excl & HDR_OFF) << HDR_OFF_SHIFT) |
                              (y0 << HDR_INIT_SHIFT) | (ovf ? HDR_POISON : 0u) | (prev ? HDR_PREV : 0u));
    // activity (reading C15) and latest PO arrival: counted once per
    // slot across overflow rounds (where prev && !ovf)
    if (!ovf && prev) {
        if (lane == 0 && total) atomicAdd(E.act_kv + (size_t)sig * (uint32_t)p.n_vdd, (unsigned long long)total);
        if (hd.z & (1u << 24)) {
            const float last = n_out ? lds_f32(E.s_out_a + 128u * (uint32_t)(n_out - 1)) : 0.0f;
            const uint32_t m = __reduce_max_sync(0xffffffffu, __float_as_uint(last));
            if (lane == 0 && m) atomicMax(p.latest + E.kv, m);
        }
    }
    __syncwarp();
}

__device__ __forceinline__ void eval_dispatch(const SweepParams& p, Env& E, const uint4 ins, const uint4 hd,
                                              const float4 d0, const float4 d1) {
    const float dl[8] = {d0.x, d0.y, d0.z, d0.w, d1.x, d1.y, d1.z, d1.w};
    switch ((hd.z >> 16) & 0xffu) {
        case 1: eval_gate<1>(p, E, ins, hd, dl); break;
        case 2: eval_gate<2>(p, E, ins, hd, dl); break;
        case 3: eval_gate<3>(p, E, ins, hd, dl); break;
        default: eval_gate<4>(p, E, ins, hd, dl); break;
    }
}

__device__ __forceinline__ void slot_group(const SweepParams& p, int64_t i, int lane, Env& E) {
    const int64_t sw = p.sw_list ? (int64_t)p.sw_list[i] : p.sw_first + i;
    E.kv = (int)(sw / p.n_pw);
    E.i = i;
    E.lane = lane;
    E.act_kv = p.act + E.kv;
    E.row = p.arena + (p.i_base + i) * p.region_bytes;
}

__device__ __forceinline__ void warp_smem(const SweepParams& p, int warp, int lane, Env& E) {
    extern __shared__ __align__(16) float smem[];
    float* s_in = smem + 4 + (size_t)warp * (size_t)(p.stage_words + 16 + 32 * (p.cstage + 1));
    E.s_in_a = static_cast<uint32_t>(__cvta_generic_to_shared(s_in));
    E.s_out_a = E.s_in_a + 4u * (uint32_t)(p.stage_words + 16) + 4u * (uint32_t)lane;
    E.bar = E.s_in_a + 4u * (uint32_t)(p.stage_words + 14);   // 8-B aligned, past any over-read
    E.phase = 0;
    if (lane == 0) mbar_init(E.bar);
    __syncwarp();
}

// Persistent level sweep (pass 0): one CTA owns one 32-slot group at a time
// and walks all levels with a CTA barrier between levels.
__global__ void __launch_bounds__(1024, 1) sweep_kernel(const SweepParams p) {
    extern __shared__ __align__(16) float smem[];
    int* ctr = reinterpret_cast<int*>(smem);             // two level counters (16-B header)
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    const int nw = blockDim.x >> 5;
    Env E;
    warp_smem(p, warp, lane, E);
    E.stride = (uint32_t)(p.pin_n_sw * p.region_bytes);
    const uint4* gd = reinterpret_cast<const uint4*>(p.gates);
    for (int64_t i = blockIdx.x; i < p.n_sw; i += gridDim.x) {
        slot_group(p, i, lane, E);
        const float4* dt = p.dtab + (int64_t)E.kv * p.n_gates * 2;
        if (threadIdx.x == 0) ctr[0] = __ldg(p.level_ptr);
        __syncthreads();
        for (int L = 0; L < p.depth; ++L) {
            const int g_end = __ldg(p.level_ptr + L + 1);
            if (p.dyn_grab) {
                // warps take gates of the level from a shared counter (load balance)
                int* c = ctr + (L & 1);
                for (;;) {
                    int gi = 0;
                    if (lane == 0) gi = atomicAdd(c, 1);
                    gi = __shfl_sync(0xffffffffu, gi, 0);
                    if (gi >= g_end) break;
                    eval_dispatch(p, E, __ldg(gd + 2 * gi), __ldg(gd + 2 * gi + 1), __ldg(dt + 2 * gi),
                                  __ldg(dt + 2 * gi + 1));
                }
                if (threadIdx.x == 0 && L + 1 < p.depth) ctr[(L + 1) & 1] = g_end;
            } else {
                for (int gi = __ldg(p.level_ptr + L) + warp; gi < g_end; gi += nw)
                    eval_dispatch(p, E, __ldg(gd + 2 * gi), __ldg(gd + 2 * gi + 1), __ldg(dt + 2 * gi),
                                  __ldg(dt + 2 * gi + 1));
            }
            fence_proxy_async_global();   // this level's stores -> next levels' TMA reads
            __syncthreads();
        }
    }
}

// Level-parallel variant for overflow reruns (few slot groups): one launch per
// level, warps take (gate, slot group) items of the level grid-wide.
__global__ void __launch_bounds__(512, 2) level_kernel(const SweepParams p, int L) {
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    Env E;
    warp_smem(p, warp, lane, E);
    E.stride = (uint32_t)(p.pin_n_sw * p.region_bytes);
    const uint4* gd = reinterpret_cast<const uint4*>(p.gates);
    const int g0 = __ldg(p.level_ptr + L);
    const int64_t items = (int64_t)(__ldg(p.level_ptr + L + 1) - g0) * p.n_sw;
    const int64_t gw = (int64_t)blockIdx.x * (blockDim.x >> 5) + warp;
    const int64_t nwarps = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t it = gw; it < items; it += nwarps) {
        const int gi = g0 + (int)(it / p.n_sw);
        const int64_t i = it % p.n_sw;
        slot_group(p, i, lane, E);
        const float4* dt = p.dtab + (int64_t)E.kv * p.n_gates * 2;
        eval_dispatch(p, E, __ldg(gd + 2 * gi), __ldg(gd + 2 * gi + 1), __ldg(dt + 2 * gi), __ldg(dt + 2 * gi + 1));
    }
    fence_proxy_async_global();   // stores -> next launch's TMA reads
}

// Materialise PI waveforms of a round's slot groups (reading C2: one event at
// t = 0 iff p1 != p2) as regions of buffers 0..n_pi-1: one warp per (PI, group).
__global__ void pi_regions_kernel(const SweepParams p, int32_t n_pi) {
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (gw >= (int64_t)n_pi * p.pin_n_sw) return;
    const int pi = (int)(gw / p.pin_n_sw);
    const int64_t i = gw % p.pin_n_sw;
    const int64_t sw = p.sw_list ? (int64_t)p.sw_list[i] : p.sw_first + i;
    const int kv = (int)(sw / p.n_pw), pw = (int)(sw % p.n_pw);
    const int64_t j = (int64_t)pw * 32 + lane;
    const int64_t pub = (int64_t)kv * p.n_pairs + j;
    const bool valid = j < p.n_pairs && pub >= p.slot_first && pub < p.slot_end;
    const uint32_t mask = __ballot_sync(0xffffffffu, valid);
    const uint32_t w1 = p.p1t[(int64_t)pi * p.n_pw + pw] & mask;
    const uint32_t w2 = p.p2t[(int64_t)pi * p.n_pw + pw] & mask;
    const uint32_t tog = w1 ^ w2;
    const uint32_t n = (tog >> lane) & 1u;
    const uint32_t off = __popc(tog & ((1u << lane) - 1u));
    uint8_t* r = p.arena + ((int64_t)pi * p.pin_n_sw + i) * p.region_bytes;
    reinterpret_cast<uint32_t*>(r)[lane] = n | (off << HDR_OFF_SHIFT) | (((w1 >> lane) & 1u) << HDR_INIT_SHIFT);
    reinterpret_cast<float*>(r + 128)[lane] = 0.0f;
}

cudaError_t launch_pi_regions(const SweepParams& p, int32_t n_pi, cudaStream_t st) {
    const int64_t threads = (int64_t)n_pi * p.pin_n_sw * 32;
    if (threads == 0) return cudaSuccess;
    pi_regions_kernel<<<(unsigned)((threads + 255) / 256), 256, 0, st>>>(p, n_pi);
    return cudaGetLastError();
}

int sweep_smem_bytes(int warps_per_cta, int stage_words, int cstage) {
    return 16 + warps_per_cta * (stage_words + 16 + 32 * (cstage + 1)) * 4;
}

cudaError_t sweep_occupancy(int warps_per_cta, int smem, int* blocks_per_sm) {
    cudaError_t e = cudaFuncSetAttribute(sweep_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, sweep_kernel, warps_per_cta * 32, smem);
}

cudaError_t launch_sweep(const SweepParams& p, int grid, int warps_per_cta, cudaStream_t st) {
    const int smem = sweep_smem_bytes(warps_per_cta, p.stage_words, p.cstage);
    cudaError_t e = cudaFuncSetAttribute(sweep_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    sweep_kernel<<<grid, warps_per_cta * 32, smem, st>>>(p);
    return cudaGetLastError();
}

cudaError_t level_occupancy(int warps_per_cta, int smem, int* blocks_per_sm) {
    cudaError_t e = cudaFuncSetAttribute(level_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, level_kernel, warps_per_cta * 32, smem);
}

cudaError_t launch_level(const SweepParams& p, int level, int grid, int warps_per_cta, cudaStream_t st) {
    const int smem = sweep_smem_bytes(warps_per_cta, p.stage_words, p.cstage);
    cudaError_t e = cudaFuncSetAttribute(level_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    level_kernel<<<grid, warps_per_cta * 32, smem, st>>>(p, level);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// H4: p[pair][words] -> pt[pi][n_pw], bit l of pt[i][w] = PI i of pair 32w+l.
// One warp per (word b, pair-group w): 32 ballots transpose a 32x32 bit block.
// ---------------------------------------------------------------------------
__global__ void expand_kernel(const uint32_t* __restrict__ p1, const uint32_t* __restrict__ p2,
                              int64_t n_pairs, int32_t words, int32_t n_pi, int32_t n_pw,
                              uint32_t* __restrict__ p1t, uint32_t* __restrict__ p2t) {
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (gw >= (int64_t)words * n_pw) return;
    const int b = (int)(gw / n_pw);
    const int pw = (int)(gw % n_pw);
    const int64_t pair = (int64_t)pw * 32 + lane;
    const uint32_t w1 = pair < n_pairs ? p1[pair * words + b] : 0u;
    const uint32_t w2 = pair < n_pairs ? p2[pair * words + b] : 0u;
    uint32_t m1 = 0, m2 = 0;
#pragma unroll 4
    for (int bit = 0; bit < 32; ++bit) {
        const uint32_t r1 = __ballot_sync(0xffffffffu, (w1 >> bit) & 1u);
        const uint32_t r2 = __ballot_sync(0xffffffffu, (w2 >> bit) & 1u);
        if (lane == bit) { m1 = r1; m2 = r2; }
    }
    const int pi = b * 32 + lane;
    if (pi < n_pi) {
        p1t[(int64_t)pi * n_pw + pw] = m1;
        p2t[(int64_t)pi * n_pw + pw] = m2;
    }
}

cudaError_t launch_expand(const uint32_t* p1, const uint32_t* p2, int64_t n_pairs, int32_t words,
                          int32_t n_pi, int32_t n_pw, uint32_t* p1t, uint32_t* p2t, cudaStream_t st) {
    const int64_t threads = (int64_t)words * n_pw * 32;
    const int bs = 256;
    const int64_t grid = (threads + bs - 1) / bs;
    if (grid == 0) return cudaSuccess;
    expand_kernel<<<(unsigned)grid, bs, 0, st>>>(p1, p2, n_pairs, words, n_pi, n_pw, p1t, p2t);
    return cudaGetLastError();
}

__device__ __forceinline__ uint32_t pair_mask(int64_t pw, int64_t lo, int64_t hi) {
    // bits l with pw*32 + l in [lo, hi)
    const int64_t a = pw * 32;
    int64_t s = lo - a, e = hi - a;
    s = s < 0 ? 0 : (s > 32 ? 32 : s);
    e = e < 0 ? 0 : (e > 32 ? 32 : e);
    if (e <= s) return 0u;
    const uint32_t upto_e = (e >= 32) ? 0xffffffffu : ((1u << e) - 1u);
    const uint32_t upto_s = (s >= 32) ? 0xffffffffu : ((1u << s) - 1u);
    return upto_e & ~upto_s;
}

// H8 for primary inputs: act[pi][k] = number of simulated pairs with p1 != p2.
__global__ void pi_activity_kernel(const uint32_t* __restrict__ p1t, const uint32_t* __restrict__ p2t,
                                   int32_t n_pi, int32_t n_pw, int64_t n_pairs, int32_t n_vdd,
                                   int64_t slot_first, int64_t slot_end, unsigned long long* act) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n_pi * n_vdd) return;
    const int pi = (int)(t / n_vdd);
    const int k = (int)(t % n_vdd);
    int64_t lo = slot_first - (int64_t)k * n_pairs, hi = slot_end - (int64_t)k * n_pairs;
    lo = lo < 0 ? 0 : lo;
    hi = hi > n_pairs ? n_pairs : hi;
    unsigned long long s = 0;
    if (hi > lo) {
        for (int64_t pw = lo / 32; pw <= (hi - 1) / 32; ++pw) {
            const uint32_t m = pair_mask(pw, lo, hi);
            s += __popc((p1t[(int64_t)pi * n_pw + pw] ^ p2t[(int64_t)pi * n_pw + pw]) & m);
        }
    }
    act[(int64_t)pi * n_vdd + k] = s;
}

cudaError_t launch_pi_activity(const uint32_t* p1t, const uint32_t* p2t, int32_t n_pi, int32_t n_pw,
                               int64_t n_pairs, int32_t n_vdd, int64_t slot_first, int64_t slot_end,
                               unsigned long long* act, cudaStream_t st) {
    const int64_t n = (int64_t)n_pi * n_vdd;
    if (n == 0) return cudaSuccess;
    pi_activity_kernel<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(p1t, p2t, n_pi, n_pw, n_pairs, n_vdd,
                                                                    slot_first, slot_end, act);
    return cudaGetLastError();
}

// H7: list the slot groups whose pass overflowed (order is irrelevant: every
// group's results are independent of where it is processed).
__global__ void compact_kernel(const int32_t* __restrict__ ovf, int64_t n_sw, const int32_t* __restrict__ sw_list,
                               int64_t sw_first, int32_t* out_list, int32_t* out_count) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n_sw || !ovf[i]) return;
    const int32_t pos = atomicAdd(out_count, 1);
    out_list[pos] = sw_list ? sw_list[i] : (int32_t)(sw_first + i);
}

cudaError_t launch_compact_overflow(const int32_t* ovf, int64_t n_sw, const int32_t* sw_list,
                                    int64_t sw_first, int32_t* out_list, int32_t* out_count,
                                    cudaStream_t st) {
    if (n_sw == 0) return cudaSuccess;
    compact_kernel<<<(unsigned)((n_sw + 255) / 256), 256, 0, st>>>(ovf, n_sw, sw_list, sw_first, out_list,
                                                                   out_count);
    return cudaGetLastError();
}

// H9: readback of kept waveforms (PIs from the stimuli, gates from the round
// that holds each slot group's final data).
__global__ void gather_kernel(const GatherParams p) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)p.n_sig * p.n_slots) return;
    const int q = (int)(t / p.n_slots);
    const int64_t s = p.slot0 + t % p.n_slots;
    const int64_t k = s / p.n_pairs, j = s % p.n_pairs;
    const int64_t pw = j / 32;
    const int lane = (int)(j % 32);
    const int64_t sw = k * p.n_pw + pw;
    const uint32_t loc = p.sig_loc[q];
    uint32_t init = 0;
    int n = 0;
    float* tout = p.times ? p.times + t * p.cap : nullptr;
    if ((loc & LOC_KIND) == LOC_PI) {
        const uint32_t w1 = p.p1t[(int64_t)(loc & LOC_ID) * p.n_pw + pw];
        const uint32_t w2 = p.p2t[(int64_t)(loc & LOC_ID) * p.n_pw + pw];
        init = (w1 >> lane) & 1u;
        n = (int)(((w1 ^ w2) >> lane) & 1u);
        if (tout && p.cap > 0) tout[0] = 0.0f;
        if (tout) for (int i = n; i < p.cap; ++i) tout[i] = 0.0f;
    } else {
        const int r = p.sw_round[sw];
        if (r < 0) { atomicOr(p.bad, 1); return; }
        const GatherRound R = p.rounds[r];
        const uint8_t* base = R.pinned + ((int64_t)(loc & LOC_ID) * R.n_sw + p.sw_index[sw]) * R.region_bytes;
        const uint32_t* hdr = reinterpret_cast<const uint32_t*>(base);
        const uint32_t h = hdr[lane];
        if (h & HDR_POISON) { atomicOr(p.bad, 2); return; }
        init = (h >> HDR_INIT_SHIFT) & 1u;
        n = (int)(h & HDR_N);
        const int off = (int)((h >> HDR_OFF_SHIFT) & HDR_OFF);
        const float* ev = reinterpret_cast<const float*>(base + 128) + off;
        if (tout) for (int i = 0; i < p.cap; ++i) tout[i] = i < n ? ev[i] : 0.0f;
    }
    p.init[t] = (uint8_t)init;
    p.count[t] = n;
}

cudaError_t launch_gather(const GatherParams& p, cudaStream_t st) {
    const int64_t n = (int64_t)p.n_sig * p.n_slots;
    if (n == 0) return cudaSuccess;
    gather_kernel<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(p);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// NEXT-1: capture / test-response analysis.  One warp per (PO, slot group):
// each lane samples its slot's PO waveform at the capture time of the slot's
// operating point (value(t) = init xor #{t_i <= t} mod 2, reading C1) and
// compares with the settled value.
// ---------------------------------------------------------------------------
__global__ void capture_kernel(const CaptureParams p) {
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (gw >= (int64_t)p.n_po * p.n_sw) return;
    const int o = (int)(gw / p.n_sw);
    const int64_t i = gw % p.n_sw;
    const int64_t sw = p.sw_lo + i;
    const int kv = (int)(sw / p.n_pw), pw = (int)(sw % p.n_pw);
    const int64_t j = (int64_t)pw * 32 + lane;
    const int64_t pub = (int64_t)kv * p.n_pairs + j;
    const bool valid = j < p.n_pairs && pub >= p.slot_first && pub < p.slot_end;
    const float T = p.t_clk[kv];
    const uint32_t loc = p.po_loc[o];
    uint32_t init = 0, n = 0, c = 0;
    float last = 0.0f;
    if ((loc & LOC_KIND) == LOC_PI) {
        const uint32_t w1 = p.p1t[(int64_t)(loc & LOC_ID) * p.n_pw + pw];
        const uint32_t w2 = p.p2t[(int64_t)(loc & LOC_ID) * p.n_pw + pw];
        init = (w1 >> lane) & 1u;
        n = ((w1 ^ w2) >> lane) & 1u;
        c = (n && 0.0f <= T) ? 1u : 0u;
    } else {
        const int r = p.sw_round[sw];
        const GatherRound R = p.rounds[r < 0 ? 0 : r];
        const uint8_t* base = R.pinned + ((int64_t)(loc & LOC_ID) * R.n_sw + p.sw_index[sw]) * R.region_bytes;
        const uint32_t h = reinterpret_cast<const uint32_t*>(base)[lane];
        init = (h >> HDR_INIT_SHIFT) & 1u;
        n = h & HDR_N;
        const float* ev = reinterpret_cast<const float*>(base + 128) + ((h >> HDR_OFF_SHIFT) & HDR_OFF);
        if (valid)
            for (uint32_t e = 0; e < n; ++e) {
                const float t = ev[e];
                last = t;
                c += (t <= T) ? 1u : 0u;
            }
    }
    const bool fail = valid && (((init ^ c) & 1u) != ((init ^ n) & 1u));
    const uint32_t fb = __ballot_sync(0xffffffffu, fail);
    if (lane == 0 && fb) atomicAdd(p.fail_po + (int64_t)o * p.n_vdd + kv, (uint32_t)__popc(fb));
    if (fail) atomicOr(p.slot_fail + i * 32 + lane, 1u);
    if (valid && last > 0.0f) atomicMax(p.slot_last + i * 32 + lane, __float_as_uint(last));
}

// per simulated slot: fail count, fail bit, slack histogram
__global__ void capture_finish_kernel(const CaptureParams p) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= p.n_sw * 32) return;
    const int64_t i = t >> 5;
    const int lane = (int)(t & 31);
    const int64_t sw = p.sw_lo + i;
    const int kv = (int)(sw / p.n_pw), pw = (int)(sw % p.n_pw);
    const int64_t j = (int64_t)pw * 32 + lane;
    const int64_t pub = (int64_t)kv * p.n_pairs + j;
    if (!(j < p.n_pairs && pub >= p.slot_first && pub < p.slot_end)) return;
    const uint32_t f = p.slot_fail[t];
    if (f) atomicAdd(p.fail_pairs + kv, 1u);
    if (p.fail_bits) p.fail_bits[pub - p.slot_first] = (uint8_t)f;
    if (p.hist) {
        const float slack = p.t_clk[kv] - __uint_as_float(p.slot_last[t]);
        int b = (int)floorf((slack - p.lo) / p.width);
        b = b < 0 ? 0 : (b >= p.n_bins ? p.n_bins - 1 : b);
        atomicAdd(p.hist + (int64_t)kv * p.n_bins + b, 1u);
    }
}

cudaError_t launch_capture(const CaptureParams& p, cudaStream_t st) {
    const int64_t threads = (int64_t)p.n_po * p.n_sw * 32;
    if (threads > 0) {
        capture_kernel<<<(unsigned)((threads + 255) / 256), 256, 0, st>>>(p);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
    }
    const int64_t t2 = p.n_sw * 32;
    if (t2 > 0) capture_finish_kernel<<<(unsigned)((t2 + 255) / 256), 256, 0, st>>>(p);
    return cudaGetLastError();
}

// NEXT-4: switching energy per operating point, warp-reduced double atomics
__global__ void energy_kernel(const unsigned long long* __restrict__ act, const double* __restrict__ c_load,
                              const double* __restrict__ vdd, const int32_t* __restrict__ island, int32_t n_isl,
                              int32_t n_pi, int32_t n_gates, int32_t n_vdd, double* out) {
    const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const double c = g < n_gates ? c_load[g] : 0.0;
    const int isl = g < n_gates ? island[g] : 0;
    for (int k = 0; k < n_vdd; ++k) {
        const double v = vdd[(size_t)k * n_isl + isl];
        double e = g < n_gates ? 0.5 * (double)act[(n_pi + g) * n_vdd + k] * c * v * v : 0.0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) e += __shfl_down_sync(0xffffffffu, e, o);
        if ((threadIdx.x & 31) == 0 && e != 0.0) atomicAdd(out + k, e);
    }
}

cudaError_t launch_energy(const unsigned long long* act, const double* c_load, const double* vdd,
                          const int32_t* island, int32_t n_isl, int32_t n_pi, int32_t n_gates, int32_t n_vdd,
                          double* out, cudaStream_t st) {
    if (n_gates <= 0) return cudaSuccess;
    energy_kernel<<<(unsigned)((n_gates + 255) / 256), 256, 0, st>>>(act, c_load, vdd, island, n_isl, n_pi, n_gates,
                                                                     n_vdd, out);
    return cudaGetLastError();
}

}  // namespace avfs
