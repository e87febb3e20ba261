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
//                           gate: delays from the FP64 delay table (P:L139,
//                           Eq. 9), coalesced header loads, an
//                           event-parallel merge + inertial filter (P:L148,
//                           readings C3-C6) built from warp ballots, compact
//                           stores, capacity check, activity and
//                           latest-arrival reductions (P:L141 step 4).
//   level_kernel        H7  the same evaluation, one launch per level, for
//                           the overflow reruns.
//   compact_kernel      H7  list of overflowed slot groups for the rerun.
//   gather_kernel       H9  readback of kept waveforms.
#include <cuda_runtime.h>
#include <cstdint>

#include "avfs_internal.h"

#ifndef AVFS_PRUNE
#define AVFS_PRUNE 1          // drop input events the gate cannot observe in that slot
#endif
#ifndef AVFS_PTX_MERGE
#define AVFS_PTX_MERGE 1      // 2-input staged merge as one PTX loop (0: the C++ loop)
#endif

namespace avfs {

// Waveforms are produced and consumed inside one launch: read them at L2
// (.cg), never through a possibly stale L1 line.
__device__ __forceinline__ uint32_t ld_u32(const void* p) {
    return __ldcg(reinterpret_cast<const unsigned int*>(p));
}
__device__ __forceinline__ float ld_f32(const void* p) { return __ldcg(reinterpret_cast<const float*>(p)); }

__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}
__device__ __forceinline__ uint32_t lanemask_le() {
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_le;" : "=r"(m));
    return m;
}

// inclusive warp prefix sum; the shuffle's in-range predicate guards the add
__device__ __forceinline__ uint32_t warp_incl_scan(uint32_t v, int) {
#pragma unroll
    for (int o = 1; o < 32; o <<= 1)
        asm("{\n .reg .pred p;\n .reg .b32 u;\n"
            " shfl.sync.up.b32 u|p, %0, %1, 0, 0xffffffff;\n"
            " @p add.u32 %0, %0, u;\n}\n" : "+r"(v) : "r"(o));
    return v;
}

#define AVFS_INF __int_as_float(0x7f800000)
#define FULL 0xffffffffu

// ---------------------------------------------------------------------------
// Gate evaluation for one gate x one 32-slot group.
//
// Lane l = slot l.  The K input header words (staged rows in shared memory,
// or one coalesced 128-B row each) give per slot the event counts n_q, the
// offsets of the event lists, the initial input values and hence the
// initial output y0 = TT(inputs) (reading C1).  m = sum_q n_q bounds the
// slot's output events; its warp prefix sum places slot l's outputs at
// offset base(l) of the output region (the header stores offset and count).
// Each lane then merges its K sorted lists (ties: ascending pin, reading C5)
// for exactly max_l m(l) steps, evaluating the truth table after every input
// event and applying the inertial filter (reading C3: a change whose
// time precedes the pending output cancels it, reading C4: no reschedule on
// confirming events); surviving outputs t + d(pin, polarity) (Eq. 9 delays)
// are stored as they are pushed -- only the last one can later be cancelled,
// and the next push overwrites it.
//
// Capacity: the region of a 32-slot group holds W = 32 C times; a gate-warp
// whose inputs carry more than W events in total (an upper bound of its
// outputs) is poisoned and the slot group rerun at 4C (reading C17).
// ---------------------------------------------------------------------------

struct Env {
    uint8_t* row;                  // arena + i * region_bytes
    uint32_t stride;               // bytes between buffers = n_sw * region_bytes (< 4 GiB, checked on host)
    int64_t i;                     // index of the slot group in the round (overflow flag)
    int kv, lane;
    unsigned long long* act_kv;    // &act[0][kv]
};

__device__ __forceinline__ uint8_t* region(uint32_t buf, const Env& E) {
    return E.row + (uint64_t)buf * (uint64_t)E.stride;
}

// First event word of a region: in place, or in the spill heap (HDR_SPILL in
// any of the region's header words; the address is the region's first
// event word pair).
__device__ __forceinline__ const uint8_t* ev_base(const uint8_t* reg, uint32_t hw) {
    const uint8_t* b = reg + 128;
    if (hw & HDR_SPILL) b = reinterpret_cast<const uint8_t*>(__ldcg(reinterpret_cast<const unsigned long long*>(b)));
    return b;
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ float lds_f32(uint32_t a) {
    float v;
    asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint32_t lds_u32(uint32_t a) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

constexpr int EV_STAGE = 256;   // staged event words per gate (EV_STAGE / K' per input)

// Where a gate's inputs are: header rows (4 x 32 words) and, if they fit, the
// inputs' compact event lists staged in shared memory by the sweep pipeline.
struct Staged {
    bool hdr, ev;
    uint32_t hdr_s;       // shared address of header row 0 (row q at + 128 q)
    uint32_t ev_s[1];     // shared address of the staged events (input q at + 4 EV_STAGE q / K')
    uint32_t dly_s;       // shared address of the gate's 8 delays [pin][pol]
    uint32_t grp_s;       // shared address of the slot group's index in the round (u32; read when poisoning)
};
__device__ __forceinline__ uint4 lds_u32x4(uint32_t a) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
    return v;
}
__device__ __forceinline__ void sts_u32(uint32_t a, uint32_t v) {
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ float4 lds_f32x4(uint32_t a) {
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(a));
    return v;
}

// Lane-serial merge + inertial filter of one slot.  Input q's list: n[q]
// events from ev[q] (shared-memory addresses if STAGED, else global
// pointers); outputs go to out[0..).  Runs exactly `steps` (= the warp's max
// m) steps; lanes with fewer events idle through the rest.  Returns the
// output count.  One step: take the earliest head (ties: lower pin), flip
// that pin, evaluate the truth table, and apply the filter.
struct MergeIn {
    uint64_t ev[KMAX];
    int n[KMAX];
    uint32_t bits, proj, tt, dly_s;
    float4 d01;           // delays of pins 0, 1: {p0 fall, p0 rise, p1 fall, p1 rise}
};

template <bool STAGED>
__device__ __forceinline__ float ld_ev(uint64_t a) {
    return STAGED ? lds_f32((uint32_t)a) : ld_f32(reinterpret_cast<const void*>(a));
}

// Address arithmetic of the list walk: 32-bit shared-memory addresses when
// STAGED, 64-bit global pointers otherwise.
template <bool STAGED> struct EvAddr { typedef uint64_t T; };
template <> struct EvAddr<true> { typedef uint32_t T; };

// The 2-input merge + inertial filter over shared-memory lists, as one PTX
// loop with in-place predicated updates (the compiled C++ loop spends ~10 of
// its ~41 instructions per step on register copies and constants).  Same
// semantics as the generic step: ties pick pin 0, a change whose time
// precedes the pending output cancels it (equality kept), outputs are stored
// as they are pushed.  steps >= 1.
__device__ __forceinline__ uint32_t merge2_smem(uint32_t a0, uint32_t e0, uint32_t a1, uint32_t e1, uint32_t bits,
                                                uint32_t proj, uint32_t tt, float4 dl, float* out, uint32_t steps) {
    float h0 = a0 < e0 ? lds_f32(a0) : AVFS_INF;
    float h1 = a1 < e1 ? lds_f32(a1) : AVFS_INF;
    a0 += 4;
    a1 += 4;
    float tl = -AVFS_INF;
    uint32_t cnt = 0, it = 0;
    asm volatile(
        "{\n"
        ".reg .pred p, ok, live, y1, chg, canc, push, more;\n"
        ".reg .f32 t, nx, dA, dB, d, co;\n"
        ".reg .b32 a, e, y, sh;\n"
        ".reg .b64 ad;\n"
        "MERGE2_%=:\n"
        "setp.lt.f32 p, %1, %0;\n"
        "min.f32 t, %0, %1;\n"
        "selp.b32 a, %3, %2, p;\n"
        "selp.b32 e, %10, %9, p;\n"
        "setp.lt.u32 ok, a, e;\n"
        "mov.f32 nx, 0f7F800000;\n"
        "@ok ld.shared.f32 nx, [a];\n"
        "@p add.u32 %3, %3, 4;\n"
        "@!p add.u32 %2, %2, 4;\n"
        "@p mov.f32 %1, nx;\n"
        "@!p mov.f32 %0, nx;\n"
        "setp.lt.f32 live, t, 0f7F800000;\n"
        "selp.b32 sh, 2, 1, p;\n"
        "@live xor.b32 %4, %4, sh;\n"
        "shr.u32 y, %11, %4;\n"
        "and.b32 y, y, 1;\n"
        "setp.ne.u32 y1, y, 0;\n"
        "selp.f32 dA, %15, %14, y1;\n"
        "selp.f32 dB, %13, %12, y1;\n"
        "selp.f32 d, dA, dB, p;\n"
        "add.rn.f32 co, t, d;\n"
        "setp.ne.and.u32 chg, y, %5, live;\n"
        "setp.gt.and.f32 canc, %6, t, chg;\n"
        "setp.le.and.f32 push, %6, t, chg;\n"
        "mul.wide.u32 ad, %7, 4;\n"
        "add.u64 ad, ad, %16;\n"
        "@push st.global.cg.f32 [ad], co;\n"
        "@push add.u32 %7, %7, 1;\n"
        "@canc sub.u32 %7, %7, 1;\n"
        "@push mov.f32 %6, co;\n"
        "@canc mov.f32 %6, 0fFF800000;\n"
        "mov.b32 %5, y;\n"
        "add.u32 %8, %8, 1;\n"
        "setp.lt.u32 more, %8, %17;\n"
        "@more bra MERGE2_%=;\n"
        "}\n"
        : "+f"(h0), "+f"(h1), "+r"(a0), "+r"(a1), "+r"(bits), "+r"(proj), "+f"(tl), "+r"(cnt), "+r"(it)
        : "r"(e0), "r"(e1), "r"(tt), "f"(dl.x), "f"(dl.y), "f"(dl.z), "f"(dl.w), "l"(out), "r"(steps)
        : "memory");
    return cnt;
}

template <int K, bool STAGED>
__device__ __forceinline__ uint32_t merge_slot(const MergeIn& M, float* out, uint32_t steps) {
    typedef typename EvAddr<STAGED>::T A;
    uint32_t bits = M.bits, proj = M.proj;
    const uint32_t tt = M.tt;
    uint32_t cnt = 0;                            // outputs kept so far (only the last can be cancelled)
    float tl = -AVFS_INF;
    auto step = [&](float t, bool live, uint32_t y, float d) {
        const float co = t + d;
        const bool change = live && y != proj;
        const bool cancel = change && tl > t;
        const bool push = change && !cancel;
        if (push) __stcg(out + cnt, co);
        cnt = cnt + (push ? 1u : 0u) - (cancel ? 1u : 0u);
        tl = push ? co : (cancel ? -AVFS_INF : tl);
        proj = y;
    };
    if (K == 1) {
        A a = (A)M.ev[0];
        const A e = a + 4 * (uint32_t)M.n[0];
        float h = a < e ? ld_ev<STAGED>(a) : AVFS_INF;
#pragma unroll 1
        for (uint32_t it = 0; it < steps; ++it) {
            const float t = h;
            a += 4;
            h = a < e ? ld_ev<STAGED>(a) : AVFS_INF;
            const bool live = t < AVFS_INF;
            bits ^= live ? 1u : 0u;
            const uint32_t y = (tt >> bits) & 1u;
            step(t, live, y, y ? M.d01.y : M.d01.x);
        }
    } else if (K == 2 && STAGED && AVFS_PTX_MERGE) {
        return steps ? merge2_smem((uint32_t)M.ev[0], (uint32_t)M.ev[0] + 4 * (uint32_t)M.n[0], (uint32_t)M.ev[1],
                                   (uint32_t)M.ev[1] + 4 * (uint32_t)M.n[1], bits, proj, tt, M.d01, out, steps)
                     : 0u;
    } else if (K == 2 && !STAGED) {
        // lists in L2: each list keeps its head and the next two elements in
        // registers, so the load feeding a comparison was issued >= 2 advances
        // of that list earlier
        A a0 = (A)M.ev[0], a1 = (A)M.ev[1];
        const A e0 = a0 + 4 * (uint32_t)M.n[0], e1 = a1 + 4 * (uint32_t)M.n[1];
        float h0 = a0 < e0 ? ld_ev<false>(a0) : AVFS_INF, g0 = a0 + 4 < e0 ? ld_ev<false>(a0 + 4) : AVFS_INF,
              f0 = a0 + 8 < e0 ? ld_ev<false>(a0 + 8) : AVFS_INF;
        float h1 = a1 < e1 ? ld_ev<false>(a1) : AVFS_INF, g1 = a1 + 4 < e1 ? ld_ev<false>(a1 + 4) : AVFS_INF,
              f1 = a1 + 8 < e1 ? ld_ev<false>(a1 + 8) : AVFS_INF;
        a0 += 12;
        a1 += 12;
#pragma unroll 1
        for (uint32_t it = 0; it < steps; ++it) {
            const bool p = h1 < h0;             // ties: pin 0 first
            const float t = fminf(h0, h1);
            const A a = p ? a1 : a0;
            const float nx = a < (p ? e1 : e0) ? ld_ev<false>(a) : AVFS_INF;
            if (p) {
                h1 = g1; g1 = f1; f1 = nx; a1 += 4;
            } else {
                h0 = g0; g0 = f0; f0 = nx; a0 += 4;
            }
            const bool live = t < AVFS_INF;
            bits ^= live ? (p ? 2u : 1u) : 0u;
            const uint32_t y = (tt >> bits) & 1u;
            step(t, live, y, p ? (y ? M.d01.w : M.d01.z) : (y ? M.d01.y : M.d01.x));
        }
    } else if (K == 2) {
        A a0 = (A)M.ev[0], a1 = (A)M.ev[1];
        const A e0 = a0 + 4 * (uint32_t)M.n[0], e1 = a1 + 4 * (uint32_t)M.n[1];
        float h0 = a0 < e0 ? ld_ev<STAGED>(a0) : AVFS_INF;
        float h1 = a1 < e1 ? ld_ev<STAGED>(a1) : AVFS_INF;
        a0 += 4;
        a1 += 4;
#pragma unroll 1
        for (uint32_t it = 0; it < steps; ++it) {
            const bool p = h1 < h0;             // ties: pin 0 first
            const float t = fminf(h0, h1);
            const A a = p ? a1 : a0;
            const float nx = a < (p ? e1 : e0) ? ld_ev<STAGED>(a) : AVFS_INF;
            h1 = p ? nx : h1;
            h0 = p ? h0 : nx;
            a1 = p ? a + 4 : a1;
            a0 = p ? a0 : a + 4;
            const bool live = t < AVFS_INF;
            bits ^= live ? (p ? 2u : 1u) : 0u;
            const uint32_t y = (tt >> bits) & 1u;
            step(t, live, y, p ? (y ? M.d01.w : M.d01.z) : (y ? M.d01.y : M.d01.x));
        }
    } else {
        float h[K];
        A a[K], e[K];
#pragma unroll
        for (int q = 0; q < K; ++q) {
            a[q] = (A)M.ev[q];
            e[q] = a[q] + 4 * (uint32_t)M.n[q];
            h[q] = a[q] < e[q] ? ld_ev<STAGED>(a[q]) : AVFS_INF;
            a[q] += 4;
        }
#pragma unroll 1
        for (uint32_t it = 0; it < steps; ++it) {
            float t = h[0];
            int pm = 0;
#pragma unroll
            for (int q = 1; q < K; ++q) {
                const bool lt = h[q] < t;
                t = lt ? h[q] : t;
                pm = lt ? q : pm;
            }
            A ap = a[0], ep = e[0];
#pragma unroll
            for (int q = 1; q < K; ++q)
                if (pm == q) { ap = a[q]; ep = e[q]; }
            const float nx = ap < ep ? ld_ev<STAGED>(ap) : AVFS_INF;
#pragma unroll
            for (int q = 0; q < K; ++q)
                if (pm == q) { h[q] = nx; a[q] = ap + 4; }
            const bool live = t < AVFS_INF;
            bits ^= live ? (1u << pm) : 0u;
            const uint32_t y = (tt >> bits) & 1u;
            step(t, live, y, lds_f32(M.dly_s + 8 * pm + 4 * y));
        }
    }
    return cnt;
}

template <int K, bool RERUN>
__device__ __forceinline__ void eval_gate(const SweepParams& p, const Env& E, const uint4 ins, const uint4 hd,
                                          const Staged& S) {
    const int lane = E.lane;
    const uint32_t out_loc = hd.x, sig = hd.y;
    const uint32_t tt = hd.z & 0xffffu;
    const uint32_t in_loc[KMAX] = {ins.x, ins.y, ins.z, ins.w};
    uint32_t hw[KMAX];
#pragma unroll
    for (int q = 0; q < K; ++q)
        hw[q] = S.hdr ? lds_u32(S.hdr_s + 128 * q + 4 * lane)
                      : __ldcg(reinterpret_cast<const uint32_t*>(region(in_loc[q], E)) + lane);
    int n[KMAX] = {0, 0, 0, 0};
    uint32_t bits = 0, orh = 0;
#pragma unroll
    for (int q = 0; q < K; ++q) {
        n[q] = (int)(hw[q] & HDR_N);
        bits |= ((hw[q] >> HDR_INIT_SHIFT) & 1u) << q;
        orh |= hw[q];
    }
    if (K == 2 && AVFS_PRUNE) {                          // table lookup (host-built, GateDesc.obs)
        const uint32_t st = (n[0] == 0 ? 1u : 0u) | (n[1] == 0 ? 2u : 0u);
        const uint32_t ob = hd.w >> (2 * (st | ((bits & st) << 2)));
        n[0] = (ob & 1u) ? n[0] : 0;
        n[1] = (ob & 2u) ? n[1] : 0;
    } else if (K >= 3 && AVFS_PRUNE) {
        // Events this slot's output cannot observe: with the stable inputs
        // (no event) at their values, the truth table restricted to the
        // remaining minterms does not depend on input q (e.g. AND with another
        // input stable at 0).  Such events never change the evaluated output
        // (reading C4), so they are dropped from the merge -- fewer merge
        // steps and tighter output offsets, identical waveforms.
        constexpr uint32_t POS[4] = {0xAAAAu, 0xCCCCu, 0xF0F0u, 0xFF00u};
        uint32_t mt = 0xFFFFu >> (16 - (1 << K));       // minterms consistent with the stable inputs
#pragma unroll
        for (int q = 0; q < K; ++q)
            if (n[q] == 0) mt &= ((bits >> q) & 1u) ? POS[q] : ~POS[q];
#pragma unroll
        for (int q = 0; q < K; ++q)
            if ((((tt >> (1 << q)) ^ tt) & mt & ~POS[q]) == 0) n[q] = 0;
    }
    int m = 0;
#pragma unroll
    for (int q = 0; q < K; ++q) m += n[q];
    const uint32_t y0 = (tt >> bits) & 1u;
    uint8_t* ro = region(out_loc, E);
    uint32_t* ro_hdr = reinterpret_cast<uint32_t*>(ro);
    auto poison = [&](bool own) {
        __stcg(ro_hdr + lane, HDR_POISON | (y0 << HDR_INIT_SHIFT));
        if (lane == 0) {            // poison bitmap bit of this (slot group, gate) in this round
            const uint32_t gi = lds_u32(S.grp_s);
            const uint64_t gbit = (uint64_t)gi * (uint32_t)p.n_gates + (sig - (uint32_t)p.n_pi);
            atomicOr(p.pois + (gbit >> 5), 1u << (gbit & 31u));
            if (own) p.ovf[gi] = 1;
        }
    };
    // one warp reduction: upstream poison, any input event
    const uint32_t R = __reduce_or_sync(FULL, (orh & HDR_POISON) | (m != 0 ? 1u : 0u));
    if (R & HDR_POISON) {                               // upstream overflow: nothing valid here
        poison(false);
        return;
    }
    if (!(R & 1u)) {                                    // no input event in any slot: constant output
        __stcg(ro_hdr + lane, y0 << HDR_INIT_SHIFT);
        return;
    }
    const uint32_t incl = warp_incl_scan((uint32_t)m, lane);
    const uint32_t total_in = __shfl_sync(FULL, incl, 31);
    const uint32_t base = incl - (uint32_t)m;
    const uint32_t maxm = __reduce_max_sync(FULL, (uint32_t)m);
    // the inputs' events bound the outputs (reading C17): header fields must
    // hold them; more than W go to the spill heap, and if the heap is
    // exhausted the slot group is rerun
    if (total_in > HDR_OFF || maxm > HDR_N) {
        poison(true);
        return;
    }
    float* out = reinterpret_cast<float*>(ro + 128) + base;
    uint32_t hdr_part = (base << HDR_OFF_SHIFT) | (y0 << HDR_INIT_SHIFT);
    if (total_in > (uint32_t)p.W) {
        const uint32_t need = (total_in + 3u) & ~3u;
        unsigned long long wb = 0;
        if (lane == 0) wb = atomicAdd(p.spill_top, (unsigned long long)need);
        wb = __shfl_sync(FULL, wb, 0);
        if (wb + need > p.spill_words) {
            poison(true);
            return;
        }
        if (lane == 0) __stcg(reinterpret_cast<unsigned long long*>(ro + 128), reinterpret_cast<unsigned long long>(p.spill + wb));
        out = p.spill + wb + base;
        hdr_part |= HDR_SPILL;
    }
    MergeIn M;
    M.bits = bits;
    M.proj = y0;
    M.tt = tt;
    M.dly_s = S.dly_s;
    if (K <= 2) M.d01 = lds_f32x4(S.dly_s);
#pragma unroll
    for (int q = 0; q < KMAX; ++q) M.n[q] = n[q];
    uint32_t my_n;
    if (S.ev) {
#pragma unroll
        for (int q = 0; q < K; ++q)
            M.ev[q] = S.ev_s[0] + (uint32_t)(4 * EV_STAGE / (K > 2 ? 4 : K)) * q + 4 * ((hw[q] >> HDR_OFF_SHIFT) & HDR_OFF);
        my_n = merge_slot<K, true>(M, out, maxm);
    } else {
#pragma unroll
        for (int q = 0; q < K; ++q)
            M.ev[q] = reinterpret_cast<uint64_t>(ev_base(region(in_loc[q], E), hw[q])) + 4 * ((hw[q] >> HDR_OFF_SHIFT) & HDR_OFF);
        my_n = merge_slot<K, false>(M, out, maxm);
    }
    __stcg(reinterpret_cast<uint32_t*>(region(out_loc, E)) + lane, my_n | hdr_part);
    // activity (reading C15) and latest PO arrival: counted once per
    // slot across rerun rounds -- only where the previous round poisoned this
    // gate of this slot group (pass 0: everywhere)
    bool prev = true;
    if (RERUN) {
        const uint64_t b = (uint64_t)__ldg(p.prev_idx + p.i_base + E.i) * (uint32_t)p.n_gates + (sig - (uint32_t)p.n_pi);
        prev = (__ldg(p.pois_prev + (b >> 5)) >> (b & 31u)) & 1u;
    }
    if (prev) {
        const uint32_t total = __reduce_add_sync(FULL, my_n);
        if (lane == 0 && total) atomicAdd(E.act_kv + (size_t)sig * (uint32_t)p.n_vdd, (unsigned long long)total);
        if (hd.z & (1u << 24)) {
            const float last = my_n ? __ldcg(out + my_n - 1) : 0.0f;
            const uint32_t mx = __reduce_max_sync(FULL, __float_as_uint(last));
            if (lane == 0 && mx) atomicMax(p.latest + E.kv, mx);
        }
    }
}

template <bool RERUN>
__device__ __forceinline__ void eval_dispatch(const SweepParams& p, const Env& E, const uint4 ins, const uint4 hd,
                                              const Staged& S) {
    // compare chain in order of frequency (2-input cells first) instead of a
    // jump table
    const uint32_t k = (hd.z >> 16) & 0xffu;
    if (k == 2) eval_gate<2, RERUN>(p, E, ins, hd, S);
    else if (k == 1) eval_gate<1, RERUN>(p, E, ins, hd, S);
    else if (k == 3) eval_gate<3, RERUN>(p, E, ins, hd, S);
    else eval_gate<4, RERUN>(p, E, ins, hd, S);
}

__device__ __forceinline__ void slot_group(const SweepParams& p, int64_t i, int lane, Env& E) {
    const int64_t sw = p.sw_list ? (int64_t)p.sw_list[i] : p.sw_first + i;
    E.kv = (int)(sw / p.n_pw);
    E.i = i;
    E.lane = lane;
    E.act_kv = p.act + E.kv;
    E.row = p.arena + (p.i_base + i) * p.region_bytes;
}

// Per-warp shared memory (words): two descriptor windows of DW gates
// (GateDesc 8 words each, then the gates' delays 8 words each), a header ring
// 4 x 128 (4 input rows of 32 header words), an event ring 2 x EV_STAGE
// (input q of a K-input gate owns EV_STAGE / K' words, K' = K rounded up to a
// power of two), staged flags.
constexpr int DW = 16;                                // gates per descriptor window
constexpr int OFF_DESC = 0, OFF_HDR = OFF_DESC + 2 * 16 * DW, OFF_EV = OFF_HDR + 4 * 128,
              OFF_META = OFF_EV + 2 * EV_STAGE;
constexpr int WARP_SMEM_WORDS = OFF_META + 4;
constexpr int LEVEL_SMEM_WORDS = 12;                  // delays of the current gate, group index

__device__ __forceinline__ float* warp_smem(int warp, int words) {
    extern __shared__ __align__(16) float smem[];
    return smem + 4 + (size_t)warp * words;
}

// Persistent level sweep (pass 0): one CTA owns one 32-slot group at a time
// and walks all levels with a CTA barrier between levels.  Warp w
// evaluates a contiguous block of each level's gates through a software
// pipeline of asynchronous copies into shared memory (cp.async): descriptors
// and delays arrive 16 gates at a time; at gate j the warp fetches the input
// header rows of gate j+2 and the input event lists of gate j+1, so the
// evaluation of gate j never waits for DRAM.  Event lists larger than the
// stage are read from L2 by the evaluation instead.
__global__ void __launch_bounds__(AVFS_SWEEP_THREADS, AVFS_SWEEP_MINB) sweep_kernel(const SweepParams p) {
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    const int nw = blockDim.x >> 5;
    Env E;
    // shared addresses only (no generic pointers into the warp's area)
    const uint32_t ws_s = smem_u32(warp_smem(0, 0)) + 4u * (uint32_t)(warp * WARP_SMEM_WORDS);
    const uint32_t s_desc = ws_s + 4 * OFF_DESC, s_hdr = ws_s + 4 * OFF_HDR, s_evr = ws_s + 4 * OFF_EV;
    const uint32_t s_grp = ws_s + 4 * (OFF_META + 2);
    E.stride = (uint32_t)(p.pin_n_sw * p.region_bytes);
    const uint4* gd = reinterpret_cast<const uint4*>(p.gates);
    // narrow netlists: the CTA walks G slot groups at once, nw / G warps each
    const int G = p.grp_per_cta, wpg = nw / G;
    const int sg = warp / wpg, wl = warp % wpg;
    for (int64_t i0 = (int64_t)blockIdx.x * G; i0 < p.n_sw; i0 += (int64_t)gridDim.x * G) {
        const int64_t i = i0 + sg;
        const bool valid = i < p.n_sw;                 // idle warps still meet every level barrier
        slot_group(p, valid ? i : i0, lane, E);
        __syncwarp();
        if (lane == 0) sts_u32(s_grp, (uint32_t)(p.i_base + (valid ? i : i0)));
        const float4* dt = p.dtab + (int64_t)E.kv * p.n_gates * 2;
        for (int L = 0; L < p.depth; ++L) {
            const int ls = __ldg(p.level_ptr + L), le = __ldg(p.level_ptr + L + 1);
            const int B = (le - ls + wpg - 1) / wpg;
            const int g0 = ls + wl * B;
            const int nj = valid ? max(0, min(B, le - g0)) : 0;
            // descriptor window k (gates g0 + 16k ..): lane copies 16 B of the
            // descriptors (lanes 0..31 = 16 gates x 2) and 16 B of the delays
            // descriptor ring of 2 DW gates (32 B each), delay ring behind it
            auto issue_win = [&](int k) {
                const int g = g0 + DW * k + (lane >> 1);
                const uint32_t w = s_desc + 32 * ((uint32_t)(DW * k + (lane >> 1)) & (2 * DW - 1)) + 16 * (lane & 1);
                if (g < le) {
                    cp_async16(w, gd + 2 * g + (lane & 1));
                    cp_async16(w + 32 * 2 * DW, dt + 2 * g + (lane & 1));
                }
            };
            auto desc_at = [&](uint32_t j) { return s_desc + 32 * (j & (2 * DW - 1)); };
            auto issue_hdr = [&](uint32_t j) {
                const uint32_t d = desc_at(j);
                const uint32_t q = (uint32_t)lane >> 3;
                if (q < ((lds_u32(d + 24) >> 16) & 0xffu))
                    cp_async16(s_hdr + 512 * (j & 3) + 128 * q + 16 * (lane & 7),
                               region(lds_u32(d + 4 * q), E) + 16 * (lane & 7));
            };
            // input q's events (extent = lane 31's offset + count) -> slot q of
            // the stage (EV_STAGE / K' words, 32 / K' lanes per input, <= 2
            // chunks of 16 B per lane); staged only if every input fits
            bool staged_next = false, staged_cur = false;
            auto issue_ev = [&](uint32_t j) {
                const uint32_t d = desc_at(j);
                const uint32_t k = (lds_u32(d + 24) >> 16) & 0xffu;
                const uint32_t sh = k > 2 ? 2u : (k > 1 ? 1u : 0u);      // log2 K'
                const uint32_t q = (uint32_t)lane >> (5 - sh), sub = (uint32_t)lane & (31u >> sh);
                uint32_t c = 0, w = 0;
                if (q < k) {
                    w = lds_u32(s_hdr + 512 * (j & 3) + 128 * q + 124);
                    c = (((w >> HDR_OFF_SHIFT) & HDR_OFF) + (w & HDR_N) + 3) >> 2;
                }
                const uint32_t cap = (uint32_t)(EV_STAGE / 4) >> sh;   // chunks per input
                const bool staged = __all_sync(FULL, c <= cap);
                staged_next = staged;
                if (staged && sub < c) {
                    const uint8_t* src = ev_base(region(lds_u32(d + 4 * q), E), w) + 16 * sub;
                    const uint32_t dst = s_evr + 4 * EV_STAGE * (j & 1) + (4 * EV_STAGE >> sh) * q + 16 * sub;
                    cp_async16(dst, src);
                    const uint32_t st = 512u >> sh;                     // bytes covered by one pass of the lanes
                    if (sub + (32u >> sh) < c) cp_async16(dst + st, src + st);
                }
            };
            if (nj > 0) {
                // prologue: descriptor windows 0, 1; header rows 0, 1; events of gate 0
                issue_win(0);
                if (nj > DW) issue_win(1);
                cp_async_commit();
                cp_async_wait_all();
                __syncwarp();
                issue_hdr(0);
                if (nj > 1) issue_hdr(1);
                cp_async_commit();
                cp_async_wait_all();
                __syncwarp();
                issue_ev(0);
                staged_cur = staged_next;
                cp_async_commit();
                const uint32_t nju = (uint32_t)nj;
#pragma unroll 1
                for (uint32_t j = 0; j < nju; ++j) {
                    cp_async_wait_all();
                    __syncwarp();
                    if (j % DW == 0 && j > 0 && j + DW < nju) issue_win((int)(j / DW) + 1);
                    if (j + 2 < nju) issue_hdr(j + 2);
                    const bool st_j = staged_cur;
                    if (j + 1 < nju) issue_ev(j + 1);
                    staged_cur = staged_next;
                    cp_async_commit();
                    const uint32_t d = desc_at(j);
                    const uint4 dv0 = lds_u32x4(d), dv1 = lds_u32x4(d + 16);
                    Staged S;
                    S.hdr = true;
                    S.hdr_s = s_hdr + 512 * (j & 3);
                    S.ev = st_j;
                    S.dly_s = d + 32 * 2 * DW;
                    S.grp_s = s_grp;
                    S.ev_s[0] = s_evr + 4 * EV_STAGE * (j & 1);
                    eval_dispatch<false>(p, E, dv0, dv1, S);
                }
            }
            // this level's stores -> the next levels' loads; with several slot
            // groups per CTA each group syncs only its own warps (named barrier)
            if (G == 1 || G > 15) __syncthreads();
            else asm volatile("bar.sync %0, %1;" ::"r"(1 + sg), "r"(32 * wpg) : "memory");
        }
    }
}

// The same sweep with each slot group shared by S = p.split co-resident CTAs
// (consecutive blocks; the grid is a multiple of S): CTA part s takes the
// s-th 1/S slice of every level, and the S parts meet at a level barrier
// made of an L2 counter per group.  Chosen when few slot groups would leave
// the last wave of CTAs mostly empty.  (A separate kernel: folding it into
// the one above changed that kernel's scheduling enough to cost 7 % on
// config 2.)
template <bool SPLIT>
__global__ void __launch_bounds__(AVFS_SWEEP_THREADS, AVFS_SWEEP_MINB) sweep_split_kernel(const SweepParams p) {
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    const int nw = blockDim.x >> 5;
    Env E;
    // shared addresses only (no generic pointers into the warp's area)
    const uint32_t ws_s = smem_u32(warp_smem(0, 0)) + 4u * (uint32_t)(warp * WARP_SMEM_WORDS);
    const uint32_t s_desc = ws_s + 4 * OFF_DESC, s_hdr = ws_s + 4 * OFF_HDR, s_evr = ws_s + 4 * OFF_EV;
    const uint32_t s_grp = ws_s + 4 * (OFF_META + 2);
    E.stride = (uint32_t)(p.pin_n_sw * p.region_bytes);
    const uint4* gd = reinterpret_cast<const uint4*>(p.gates);
    // narrow netlists: the CTA walks G slot groups at once, nw / G warps each;
    // few slot groups: S co-resident CTAs (consecutive blocks, grid a multiple
    // of S) share one group, each taking 1/S of every level (G == 1 then)
    const int G = SPLIT ? 1 : p.grp_per_cta, wpg = nw / G, S = SPLIT ? p.split : 1;
    const int sg = warp / wpg, wl = warp % wpg;
    const int64_t u_end = SPLIT ? p.n_sw * S : p.n_sw;
    const int64_t u_step = SPLIT ? (int64_t)gridDim.x : (int64_t)gridDim.x * G;
    for (int64_t u = SPLIT ? (int64_t)blockIdx.x : (int64_t)blockIdx.x * G; u < u_end; u += u_step) {
        const int64_t i0 = SPLIT ? u / S : u;
        const int part = SPLIT ? (int)(u % S) : 0;
        const int64_t i = i0 + sg;
        const bool valid = i < p.n_sw;                 // idle warps still meet every level barrier
        slot_group(p, valid ? i : i0, lane, E);
        __syncwarp();
        if (lane == 0) sts_u32(s_grp, (uint32_t)(p.i_base + (valid ? i : i0)));
        const float4* dt = p.dtab + (int64_t)E.kv * p.n_gates * 2;
        for (int L = 0; L < p.depth; ++L) {
            const int ls0 = __ldg(p.level_ptr + L), le0 = __ldg(p.level_ptr + L + 1);
            const int P = SPLIT ? (le0 - ls0 + S - 1) / S : 0;
            const int ls = SPLIT ? min(le0, ls0 + part * P) : ls0;
            const int le = SPLIT ? min(le0, ls + P) : le0;
            const int B = (le - ls + wpg - 1) / wpg;
            const int g0 = ls + wl * B;
            const int nj = valid ? max(0, min(B, le - g0)) : 0;
            // descriptor window k (gates g0 + 16k ..): lane copies 16 B of the
            // descriptors (lanes 0..31 = 16 gates x 2) and 16 B of the delays
            // descriptor ring of 2 DW gates (32 B each), delay ring behind it
            auto issue_win = [&](int k) {
                const int g = g0 + DW * k + (lane >> 1);
                const uint32_t w = s_desc + 32 * ((uint32_t)(DW * k + (lane >> 1)) & (2 * DW - 1)) + 16 * (lane & 1);
                if (g < le) {
                    cp_async16(w, gd + 2 * g + (lane & 1));
                    cp_async16(w + 32 * 2 * DW, dt + 2 * g + (lane & 1));
                }
            };
            auto desc_at = [&](uint32_t j) { return s_desc + 32 * (j & (2 * DW - 1)); };
            auto issue_hdr = [&](uint32_t j) {
                const uint32_t d = desc_at(j);
                const uint32_t q = (uint32_t)lane >> 3;
                if (q < ((lds_u32(d + 24) >> 16) & 0xffu))
                    cp_async16(s_hdr + 512 * (j & 3) + 128 * q + 16 * (lane & 7),
                               region(lds_u32(d + 4 * q), E) + 16 * (lane & 7));
            };
            // input q's events (extent = lane 31's offset + count) -> slot q of
            // the stage (EV_STAGE / K' words, 32 / K' lanes per input, <= 2
            // chunks of 16 B per lane); staged only if every input fits
            bool staged_next = false, staged_cur = false;
            auto issue_ev = [&](uint32_t j) {
                const uint32_t d = desc_at(j);
                const uint32_t k = (lds_u32(d + 24) >> 16) & 0xffu;
                const uint32_t sh = k > 2 ? 2u : (k > 1 ? 1u : 0u);      // log2 K'
                const uint32_t q = (uint32_t)lane >> (5 - sh), sub = (uint32_t)lane & (31u >> sh);
                uint32_t c = 0, w = 0;
                if (q < k) {
                    w = lds_u32(s_hdr + 512 * (j & 3) + 128 * q + 124);
                    c = (((w >> HDR_OFF_SHIFT) & HDR_OFF) + (w & HDR_N) + 3) >> 2;
                }
                const uint32_t cap = (uint32_t)(EV_STAGE / 4) >> sh;   // chunks per input
                const bool staged = __all_sync(FULL, c <= cap);
                staged_next = staged;
                if (staged && sub < c) {
                    const uint8_t* src = ev_base(region(lds_u32(d + 4 * q), E), w) + 16 * sub;
                    const uint32_t dst = s_evr + 4 * EV_STAGE * (j & 1) + (4 * EV_STAGE >> sh) * q + 16 * sub;
                    cp_async16(dst, src);
                    const uint32_t st = 512u >> sh;                     // bytes covered by one pass of the lanes
                    if (sub + (32u >> sh) < c) cp_async16(dst + st, src + st);
                }
            };
            if (nj > 0) {
                // prologue: descriptor windows 0, 1; header rows 0, 1; events of gate 0
                issue_win(0);
                if (nj > DW) issue_win(1);
                cp_async_commit();
                cp_async_wait_all();
                __syncwarp();
                issue_hdr(0);
                if (nj > 1) issue_hdr(1);
                cp_async_commit();
                cp_async_wait_all();
                __syncwarp();
                issue_ev(0);
                staged_cur = staged_next;
                cp_async_commit();
                const uint32_t nju = (uint32_t)nj;
#pragma unroll 1
                for (uint32_t j = 0; j < nju; ++j) {
                    cp_async_wait_all();
                    __syncwarp();
                    if (j % DW == 0 && j > 0 && j + DW < nju) issue_win((int)(j / DW) + 1);
                    if (j + 2 < nju) issue_hdr(j + 2);
                    const bool st_j = staged_cur;
                    if (j + 1 < nju) issue_ev(j + 1);
                    staged_cur = staged_next;
                    cp_async_commit();
                    const uint32_t d = desc_at(j);
                    const uint4 dv0 = lds_u32x4(d), dv1 = lds_u32x4(d + 16);
                    Staged S;
                    S.hdr = true;
                    S.hdr_s = s_hdr + 512 * (j & 3);
                    S.ev = st_j;
                    S.dly_s = d + 32 * 2 * DW;
                    S.grp_s = s_grp;
                    S.ev_s[0] = s_evr + 4 * EV_STAGE * (j & 1);
                    eval_dispatch<false>(p, E, dv0, dv1, S);
                }
            }
            // this level's stores -> the next levels' loads; with several slot
            // groups per CTA each group syncs only its own warps (named barrier)
            if (G == 1 || G > 15) __syncthreads();
            else asm volatile("bar.sync %0, %1;" ::"r"(1 + sg), "r"(32 * wpg) : "memory");
            if (SPLIT) {                                // the other parts of this level (L2 counter)
                if (threadIdx.x == 0) {
                    unsigned int* ctr = p.lvl_sync + i;
                    __threadfence();
                    atomicAdd(ctr, 1u);
                    const unsigned int target = (unsigned int)S * (unsigned int)(L + 1);
                    unsigned int v;
                    while (true) {
                        asm volatile("ld.acquire.gpu.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
                        if (v >= target) break;
                        __nanosleep(64);
                    }
                    __threadfence();
                }
                __syncthreads();
            }
        }
    }
}

// Level-parallel variant for overflow reruns (few slot groups): one launch per
// level, warps take (gate, slot group) items of the level grid-wide.
__global__ void __launch_bounds__(512, 2) level_kernel(const SweepParams p, int L) {
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    Env E;
    float* ws = warp_smem(warp, LEVEL_SMEM_WORDS);
    E.stride = (uint32_t)(p.pin_n_sw * p.region_bytes);
    const uint4* gd = reinterpret_cast<const uint4*>(p.gates);
    Staged S;
    S.hdr = false;
    S.ev = false;
    S.dly_s = smem_u32(ws);
    S.grp_s = smem_u32(ws + 8);
    const int g0 = __ldg(p.level_ptr + L);
    const int64_t items = (int64_t)(__ldg(p.level_ptr + L + 1) - g0) * p.n_sw;
    const int64_t gw = (int64_t)blockIdx.x * (blockDim.x >> 5) + warp;
    const int64_t nwarps = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t it = gw; it < items; it += nwarps) {
        const int gi = g0 + (int)(it / p.n_sw);
        const int64_t i = it % p.n_sw;
        slot_group(p, i, lane, E);
        const float* dt = reinterpret_cast<const float*>(p.dtab) + ((int64_t)E.kv * p.n_gates + gi) * 8;
        __syncwarp();
        if (lane < 8) ws[lane] = __ldg(dt + lane);
        if (lane == 8) reinterpret_cast<uint32_t*>(ws)[8] = (uint32_t)(p.i_base + i);
        __syncwarp();
        eval_dispatch<true>(p, E, __ldg(gd + 2 * gi), __ldg(gd + 2 * gi + 1), S);
    }
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

int sweep_smem_bytes(int warps_per_cta) { return 16 + warps_per_cta * WARP_SMEM_WORDS * 4; }
int level_smem_bytes(int warps_per_cta) { return 16 + warps_per_cta * LEVEL_SMEM_WORDS * 4; }

cudaError_t sweep_occupancy(int warps_per_cta, int smem, int* blocks_per_sm) {
    int b1 = 0, b2 = 0;
    cudaError_t e = cudaFuncSetAttribute(sweep_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e == cudaSuccess) e = cudaFuncSetAttribute(sweep_split_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b1, sweep_kernel, warps_per_cta * 32, smem);
    if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b2, sweep_split_kernel<true>, warps_per_cta * 32, smem);
    *blocks_per_sm = b1 < b2 ? b1 : b2;      // split groups need every CTA resident
    return e;
}

cudaError_t launch_sweep(const SweepParams& p, int grid, int warps_per_cta, cudaStream_t st) {
    const int smem = sweep_smem_bytes(warps_per_cta);
    if (p.split > 1) {
        // the parts of a slot group wait for each other: a cooperative launch
        // guarantees that every CTA of the grid is resident (or fails)
        SweepParams q = p;
        void* args[] = {&q};
        return cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(sweep_split_kernel<true>), dim3(grid),
                                           dim3(warps_per_cta * 32), args, (size_t)smem, st);
    }
    sweep_kernel<<<grid, warps_per_cta * 32, smem, st>>>(p);
    return cudaGetLastError();
}

cudaError_t level_occupancy(int warps_per_cta, int smem, int* blocks_per_sm) {
    cudaError_t e = cudaFuncSetAttribute(level_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, level_kernel, warps_per_cta * 32, smem);
}

cudaError_t launch_level(const SweepParams& p, int level, int grid, int warps_per_cta, cudaStream_t st) {
    const int smem = level_smem_bytes(warps_per_cta);
    cudaError_t e = cudaFuncSetAttribute(level_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    level_kernel<<<grid, warps_per_cta * 32, smem, st>>>(p, level);
    return cudaGetLastError();
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
                               int64_t sw_first, int32_t* out_list, int32_t* out_prev, int32_t* out_count) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n_sw || !ovf[i]) return;
    const int32_t pos = atomicAdd(out_count, 1);
    out_list[pos] = sw_list ? sw_list[i] : (int32_t)(sw_first + i);
    out_prev[pos] = (int32_t)i;
}

cudaError_t launch_compact_overflow(const int32_t* ovf, int64_t n_sw, const int32_t* sw_list,
                                    int64_t sw_first, int32_t* out_list, int32_t* out_prev,
                                    int32_t* out_count, cudaStream_t st) {
    if (n_sw == 0) return cudaSuccess;
    compact_kernel<<<(unsigned)((n_sw + 255) / 256), 256, 0, st>>>(ovf, n_sw, sw_list, sw_first, out_list,
                                                                   out_prev, out_count);
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
        const float* ev = reinterpret_cast<const float*>(ev_base(base, h)) + off;
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
        const float* ev = reinterpret_cast<const float*>(ev_base(base, h)) + ((h >> HDR_OFF_SHIFT) & HDR_OFF);
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
