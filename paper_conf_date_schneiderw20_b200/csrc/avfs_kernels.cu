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
//   expand_groups_kernel H4 the same per (PI, pair-major slot group): the PI
//                           waveforms the sweep reads (no PI storage).
//   sweep_kernel        H6+H7 persistent level sweep over slot groups
//                           (pair-major: a group's lanes are one stimulus
//                           pair's operating points), a barrier per group
//                           between levels.  Per batch of gates a
//                           bit-parallel phase (lane = gate, 32 slots per
//                           word: initial values, observable-event masks)
//                           and a per-gate pass (lane = slot: merge of the
//                           input lists with the inertial filter, P:L148,
//                           readings C3-C6).  Delays from the FP64 delay
//                           table (Eq. 9) or evaluated in the
//                           sweep.  Reruns (H7) use the same kernel on the
//                           overflowed slot groups.
//   delay_kernel        H2/H3 Eq. (4)/(9) in FP64 per (Vdd, gate, arc).
//   compact_kernel      H7  list of overflowed slot groups for the rerun.
//   gather_kernel       H9  readback of kept waveforms.
//   capture_kernel      NEXT-1 test-response analysis.
//   energy_kernel       NEXT-4 switching energy.
#include <cuda_runtime.h>
#include <cstdint>

#include "avfs_internal.h"

// Debug builds (-DAVFS_CHECKS): device asserts on the sweep's storage
// invariants -- an observable input has an entry and at least one event in
// the slot, a gate's outputs stay inside the extent reserved for it (region
// or heap allocation), heap allocations inside the heap.  A failed assert
// traps the kernel (sticky CUDA error).  scripts/gpu_checks.sh runs the GPU
// test suite on such a build.
#ifdef AVFS_CHECKS
#include <cassert>
#define AVFS_CHECK(c) assert(c)
#else
#define AVFS_CHECK(c) ((void)0)
#endif


namespace avfs {

// Byte offset of a region's in-place times (record mask A = the slots that
// own an entry): at the 128-B line after the (at most 32) entries, so that
// with line-aligned regions the times start on a line (config 4 61.5 vs
// 62.0 ms packed), or right after the popc(A) entry words
// (AVFS_TIMES_PACKED).
#ifndef AVFS_REG_GROUP_MAJOR
#define AVFS_REG_GROUP_MAJOR 1     // regions [group][buffer] (1) or [buffer][group] (0)
#endif
#ifndef AVFS_REC_GROUP_MAJOR
#define AVFS_REC_GROUP_MAJOR 1     // records [group][buffer] (1) or [buffer][group] (0)
#endif
#ifndef AVFS_TIMES_PACKED
#define AVFS_TIMES_PACKED 0        // 1: times right after the popc(A) entries; 0: at AVFS_TIMES_AT (a line boundary)
#endif
#ifndef AVFS_TIMES_AT
#define AVFS_TIMES_AT 128u         // (AVFS_TIMES_PACKED 0) fixed byte offset of a region's times: the line after 32 entries
#endif
__host__ __device__ __forceinline__ uint32_t times_off(uint32_t A) {
#if AVFS_TIMES_PACKED
#ifdef __CUDA_ARCH__
    return 4u * (uint32_t)__popc(A);
#else
    return 4u * (uint32_t)__builtin_popcount(A);
#endif
#else
    (void)A;
    return AVFS_TIMES_AT;
#endif
}

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
// Persistent level sweep (H6 + H7).
//
// A CTA walks one or more 32-slot groups at a time (pair-major: a group's
// lanes are mostly one stimulus pair at 32 operating points)
// through every level of the netlist, with a (named) barrier per group
// between levels (P:L166 level-wise processing).  A warp repeatedly grabs a
// batch of up to QN gates of the current level and evaluates it in two
// phases:
//
//  Phase A (lane = gate; bit-parallel over the 32 slots).  Each lane reads
//  its gate's descriptor and the records of the gate's inputs (init, event
//  and entry masks, counts), evaluates the truth table on the 32 initial
//  values at once (Shannon expansion, y0 = TT(inputs), reading C1) and, per
//  input q, the mask O_q of slots where q's events are observable: the
//  output is not constant over the input values the slot can take (an input
//  without events is fixed at its value, one with events is free) -- an
//  event the gate cannot observe never changes the evaluated output
//  (reading C4) and is not merged.  A = the union of the O_q.  Gates with
//  A = 0 are finished here: their record {y0, no events} is written and
//  nothing else is read.  The others are queued (shared memory) with their
//  masks, input entry / time bases and the addresses the per-gate pass
//  needs.  Time storage: a gate whose inputs carry U events in total (an
//  upper bound of its outputs, reading C17) stores its times in place if
//  U <= W, else in the round's spill heap (one bump allocation per warp);
//  heap exhausted -> poisoned and the slot group rerun (H7).
//
//  Phase B (one queued gate per pass, lane = slot).  Per lane: the slot's
//  input values and observable inputs, the entries (count, offset) of the
//  first two observable inputs, the two pins' delays at the lane's operating
//  point (delay table, or Eq. (4)/(9) evaluated here), the output offset,
//  then the lane-serial merge of the sorted input lists by (time, pin)
//  (ties: ascending pin, reading C5) with the inertial filter (
//  reading C3: a change whose time precedes the pending output cancels it,
//  equality kept; C4: no reschedule on confirming events).  Surviving
//  outputs t + d(pin, polarity) are stored as they are pushed -- only the
//  last one can later be cancelled.  Then the slot's entry, its activity
//  (reading C15, one u64 reduction per lane), a PO's latest time
//  and -- lane 0 -- the gate's record.
// ---------------------------------------------------------------------------

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
__device__ __forceinline__ uint32_t lds_u16(uint32_t a) {
    unsigned short v;
    asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ unsigned long long lds_u64(uint32_t a) {
    unsigned long long v;
    asm volatile("ld.shared.u64 %0, [%1];" : "=l"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint4 lds_u32x4(uint32_t a) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
    return v;
}
__device__ __forceinline__ float4 lds_f32x4(uint32_t a) {
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(a));
    return v;
}
__device__ __forceinline__ void sts_u32(uint32_t a, uint32_t v) {
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void sts_u16(uint32_t a, uint32_t v) {
    asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "h"((unsigned short)v) : "memory");
}
__device__ __forceinline__ void sts_u64(uint32_t a, unsigned long long v) {
    asm volatile("st.shared.u64 [%0], %1;" ::"r"(a), "l"(v) : "memory");
}
__device__ __forceinline__ void sts_u32x4(uint32_t a, uint4 v) {
    asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                 : "memory");
}
__device__ __forceinline__ void sts_f32x4(uint32_t a, float4 v) {
    asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(a), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w)
                 : "memory");
}
__device__ __forceinline__ uint32_t atoms_add(uint32_t a, uint32_t v) {
    uint32_t r;
    asm volatile("atom.shared.add.u32 %0, [%1], %2;" : "=r"(r) : "r"(a), "r"(v) : "memory");
    return r;
}
__device__ __forceinline__ void atoms_or(uint32_t a, uint32_t v) {
    asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void atoms_max(uint32_t a, uint32_t v) {
    asm volatile("red.shared.max.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void atoms_add_u64(uint32_t a, unsigned long long v) {
    asm volatile("red.shared.add.u64 [%0], %1;" ::"r"(a), "l"(v) : "memory");
}

// Debug-only phase timing (-DAVFS_PROF_PHASES): per-warp clock64 sums per
// phase, read back with avfs_debug_phase_cycles.
#ifdef AVFS_PROF_PHASES
__device__ unsigned long long g_phase_cycles[16];
#define PROF_T0() long long prof_t0_ = clock64()
#define PROF_ACC(k) do { long long t_ = clock64(); if ((threadIdx.x & 31) == 0) atomicAdd(&g_phase_cycles[k], (unsigned long long)(t_ - prof_t0_)); prof_t0_ = t_; } while (0)
#else
#define PROF_T0() do {} while (0)
#define PROF_ACC(k) do {} while (0)
#endif

#ifndef AVFS_QN
#define AVFS_QN 32
#endif
#ifndef AVFS_MIN_BATCH
#define AVFS_MIN_BATCH 12          // smallest guided / tail batch (fewer bit-parallel phases per level)
#endif
#ifndef AVFS_TAIL_SPLIT
#define AVFS_TAIL_SPLIT 1
#endif
constexpr int QN = AVFS_QN;            // gates per batch (Phase A lanes, queue entries)
constexpr int QW = 44;                 // words per queue entry
enum : int {
    Q_TTK = 0, Q_SIG = 1, Q_OUT = 2, Q_Y0 = 3,      // descriptor words, output initial values
    Q_A = 4, Q_GATE = 5, Q_FLAG = 6,                // entry mask, gate index, flags | fanout << 8
    Q_DROW = 7,                                     // the gate's delay-table row: gate x 4 x box.nk (float2 units)
    Q_TB = 8,                                       // u64 time base of the output
    Q_AROW = 10,                                    // the output's activity row: signal x n_vdd + box.k0
    Q_UNI = 11,                                     // every slot of A alike: UNI_ALIKE | fields below, else 0
    Q_X = 12, Q_E = 16, Q_AQ = 20,                  // per input: init, observable-event, entry masks
    Q_ENTB = 24,                                    // 4 x u64 entry bases of the inputs (PIs: the PI entry table)
    Q_ITB = 32,                                     // 4 x u64 time bases of the inputs
    Q_OREG = 40,                                    // u64 output region (its entries)
    Q_CAP = 42                                      // (AVFS_CHECKS) words reserved for the output's times
};
// Q_UNI: bits 0-3 the slots' input values, 4-7 their inputs with observable events
constexpr uint32_t UNI_ALIKE = 0x100u;
constexpr uint32_t QF_POISON = 1u, QF_COUNT = 2u, QF_OWN = 4u, QF_SPILL = 8u;
constexpr int WARP_INFO_WORDS = 16;  // per warp, after its queue: enc, region row, record row, gi, sw (u64 each), vmask
constexpr int WARP_SMEM_WORDS = QN * QW + WARP_INFO_WORDS;
constexpr uint32_t WS_OFF = 4u * QN * QW;          // byte offset of the warp info block from the warp's queue
constexpr int CTA_HDR_WORDS = 2 * 32 + 4;                          // level counters [group][2], pad

// A warp's slot group.  Its region and record rows (64-bit pointers) are
// kept in the warp's shared info block and loaded where used (ws), not held
// in registers through the sweep's loops.
// (warp info block at q_s + WS_OFF: +0 enc, +8 region row, +16 record row,
// +24 group index in the round, +32 slot group in the box, +40 vmask; at a
// constant offset from the warp's queue, so its loads need no address math)
struct Grp {
    uint32_t q;            // the warp's queue (shared address)
    int krel;              // this lane's operating point - box.k0
};

__device__ __forceinline__ uint8_t* grp_row(const Grp& G) { return reinterpret_cast<uint8_t*>(lds_u64(G.q + WS_OFF + 8)); }
__device__ __forceinline__ uint4* grp_rec(const Grp& G) { return reinterpret_cast<uint4*>(lds_u64(G.q + WS_OFF + 16)); }
__device__ __forceinline__ int64_t grp_gi(const Grp& G) { return (int64_t)lds_u64(G.q + WS_OFF + 24); }
__device__ __forceinline__ int64_t grp_sw(const Grp& G) { return (int64_t)lds_u64(G.q + WS_OFF + 32); }
__device__ __forceinline__ uint32_t grp_vmask(const Grp& G) { return lds_u32(G.q + WS_OFF + 40); }
// bytes between a group's arena buffers / records between its buffers
#if AVFS_REG_GROUP_MAJOR
#define GRP_STRIDE(p) ((uint32_t)(p).region_bytes)
#else
#define GRP_STRIDE(p) ((uint32_t)((p).pin_n_sw * (p).region_bytes))
#endif
#if AVFS_REC_GROUP_MAJOR
#define GRP_RSTRIDE(p) 1u
#else
#define GRP_RSTRIDE(p) ((uint32_t)(p).pin_n_sw)
#endif

// lane's slot of group sw in the box (SlotBox, avfs_internal.h): pair j,
// operating point k; false outside the box or the simulated range
__device__ __forceinline__ bool box_slot(const SlotBox& b, int64_t sw, int lane, int64_t& j, int& k) {
    const int64_t i = sw * 32 + lane;
    j = 0;
    k = b.k0;
    if (i >= b.nj * b.nk) return false;
    j = b.j0 + i / b.nk;
    if (j >= b.n_pairs) j -= b.n_pairs;
    k = b.k0 + (int)(i % b.nk);
    const int64_t pub = (int64_t)k * b.n_pairs + j;
    return pub >= b.slot_first && pub < b.slot_end;
}

__device__ __forceinline__ void group_setup(const SweepParams& p, int64_t i, int lane, Grp& G) {
    const int64_t sw = p.sw_list ? (int64_t)p.sw_list[i] : p.sw_first + i;
    const int64_t gi = p.i_base + i;
#if AVFS_REG_GROUP_MAJOR
    uint8_t* row = p.arena + gi * p.n_buf * p.region_bytes;
#else
    uint8_t* row = p.arena + gi * p.region_bytes;
#endif
#if AVFS_REC_GROUP_MAJOR
    uint4* rec = p.recs + gi * (int64_t)p.n_buf;
#else
    uint4* rec = p.recs + gi;
#endif
    int64_t j;
    int k;
    const uint32_t vmask = __ballot_sync(FULL, box_slot(p.box, sw, lane, j, k));
    G.krel = k - p.box.k0;
    if (lane == 0) {
        sts_u64(G.q + WS_OFF + 8, reinterpret_cast<unsigned long long>(row));
        sts_u64(G.q + WS_OFF + 16, reinterpret_cast<unsigned long long>(rec));
        sts_u64(G.q + WS_OFF + 24, (unsigned long long)gi);
        sts_u64(G.q + WS_OFF + 32, (unsigned long long)sw);
        sts_u32(G.q + WS_OFF + 40, vmask);
    }
    __syncwarp();
}

// all-ones iff truth-table bit b is set
__device__ __forceinline__ uint32_t tt_leaf(uint32_t tt, int b) {
    return (uint32_t)((int32_t)(tt << (31 - b)) >> 31);
}
__device__ __forceinline__ uint32_t mux(uint32_t s, uint32_t one, uint32_t zero) { return (s & one) | (~s & zero); }

// Bit-parallel gate evaluation over the 32 slots of a group.  KM = number of
// input positions evaluated (2 or 4; missing inputs have X = E = 0).
//   y0   = TT(X)                           (value before t = 0)
//   A    = can0 & can1: slots whose output is not constant over the inputs'
//          possible values (X fixed where E = 0, free where E = 1)
template <int KM>
__device__ __forceinline__ void eval_masks(uint32_t tt, const uint32_t (&X)[4], const uint32_t (&E)[4], uint32_t& y0,
                                           uint32_t& A, uint32_t (&O)[4]) {
    uint32_t lf[1 << KM];
#pragma unroll
    for (int b = 0; b < (1 << KM); ++b) lf[b] = tt_leaf(tt, b);
    uint32_t n[1 << KM];
#pragma unroll
    for (int b = 0; b < (1 << KM); ++b) n[b] = lf[b];
#pragma unroll
    for (int q = 0; q < KM; ++q)
#pragma unroll
        for (int b = 0; b < (1 << (KM - 1 - q)); ++b) n[b] = mux(X[q], n[2 * b + 1], n[2 * b]);
    y0 = n[0];
    uint32_t cons[1 << KM];
    cons[0] = E[0] | ~X[0];
    cons[1] = E[0] | X[0];
#pragma unroll
    for (int q = 1; q < KM; ++q) {
        const uint32_t l0 = E[q] | ~X[q], l1 = E[q] | X[q];
#pragma unroll
        for (int b = (1 << q) - 1; b >= 0; --b) {
            cons[b + (1 << q)] = cons[b] & l1;
            cons[b] = cons[b] & l0;
        }
    }
    // O[q]: slots where input q has events and the truth table restricted to
    // the consistent input vectors depends on q (its events are observable)
#pragma unroll
    for (int q = 0; q < 4; ++q) O[q] = 0;
#pragma unroll
    for (int q = 0; q < KM; ++q) {
        const uint32_t dq = tt ^ (tt >> (1 << q));     // bit b (b_q = 0): output differs when q toggles
        uint32_t o = 0;
#pragma unroll
        for (int b = 0; b < (1 << KM); ++b)
            if (!((b >> q) & 1)) o |= cons[b] & tt_leaf(dq, b);
        O[q] = o & E[q];
    }
    A = O[0] | O[1] | O[2] | O[3];
}

// Eq. (4) by nested Horner in FP64 with FMA, outer in x = phi_V(v) from
// i = deg_v down, inner in z = phi_C(c), then
// Eq. (9) d' = d_nom (1 + f), Q-mode rounding (reading C12), one rounding to
// binary32 (reading C11).  cf: [deg_v+1][deg_c+1].
__device__ __forceinline__ float arc_delay(const double* __restrict__ cf, int dv, int dc, double x, double z,
                                           double dnom, double q, bool& bad) {
    double f = 0.0;
    for (int i = dv; i >= 0; --i) {
        const double* row = cf + i * (dc + 1);
        double a = __ldg(row + dc);
        for (int j = dc - 1; j >= 0; --j) a = fma(a, z, __ldg(row + j));
        f = (i == dv) ? a : fma(f, x, a);
    }
    double d = dnom * (1.0 + f);
    if (q > 0.0) d = q * rint(d / q);
    bad = !(d > 0.0);
    return __double2float_rn(d);
}

__device__ __forceinline__ void poison_bit(const SweepParams& p, int64_t gi, uint32_t sig) {
    const uint64_t gbit = (uint64_t)gi * (uint32_t)p.n_gates + (sig - (uint32_t)p.n_pi);
    atomicOr(p.pois + (gbit >> 5), 1u << (gbit & 31u));
}

#ifndef AVFS_PF_L2
#define AVFS_PF_L2 1
#endif
// bulk L2 prefetch of [p, p + bytes) (16-B granules, at most AVFS_PF_MAX bytes)
#ifndef AVFS_PF_MAX
#define AVFS_PF_MAX 1024u
#endif
__device__ __forceinline__ void l2_prefetch(const void* p, uint32_t bytes) {
    const uintptr_t a = reinterpret_cast<uintptr_t>(p) & ~uintptr_t(15);
    const uint32_t n = min((bytes + 15u + (uint32_t)(reinterpret_cast<uintptr_t>(p) & 15u)) & ~15u, AVFS_PF_MAX);
    if (n) asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a), "r"(n) : "memory");
}

// Phase A for gates g0 .. g0 + nb - 1 (nb <= QN); returns the number queued.
template <bool RERUN>
__device__ __forceinline__ int phase_a(const SweepParams& p, const Grp& G, int g0, int nb, uint32_t q_s, int lane) {
    const bool on = lane < nb;
    const int g = g0 + (on ? lane : 0);
    const uint4* gd = reinterpret_cast<const uint4*>(p.gates);
    uint4 d0 = make_uint4(0, 0, 0, 0), d1 = make_uint4(0, 0, 0, 0);
    if (on) {
        d0 = __ldg(gd + 2 * g);
        d1 = __ldg(gd + 2 * g + 1);
    }
    const uint32_t tt = d1.z & 0xffffu, K = on ? (d1.z >> 16) & 0xffu : 0u;
    const uint32_t loc[4] = {d0.x, d0.y, d0.z, d0.w};
    uint32_t X[4], E[4], AQ[4], M[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        X[q] = E[q] = AQ[q] = M[q] = 0;
        if ((uint32_t)q < K) {
            const uint32_t id = loc[q] & LOC_ID;
            if ((loc[q] & LOC_KIND) == LOC_PI) {       // reading C2: one event at t = 0 iff p1 != p2
#if AVFS_PI_GMAJOR
                // the group's (p1, p2) words of every PI are one contiguous
                // block (L2-resident while the group is swept)
                const uint2 pw = __ldg(reinterpret_cast<const uint2*>(p.p1g) + (grp_sw(G) * p.n_pi + id));
                const uint32_t w1 = pw.x, w2 = pw.y;
#else
                const int64_t ix = (int64_t)id * p.n_grp + grp_sw(G);
                const uint32_t w1 = __ldg(p.p1g + ix), w2 = __ldg(p.p2g + ix);
#endif
                X[q] = w1;
                E[q] = AQ[q] = (w1 ^ w2) & grp_vmask(G);
                M[q] = (uint32_t)__popc(E[q]);
            } else {
                const uint4 r = __ldcg(grp_rec(G) + (size_t)id * GRP_RSTRIDE(p));
                X[q] = r.x;
                E[q] = r.y;
                AQ[q] = r.z;
                M[q] = r.w;
            }
        }
    }
    uint32_t y0, A, O[4];
    if (__any_sync(FULL, K > 2)) eval_masks<4>(tt, X, E, y0, A, O);
    else eval_masks<2>(tt, X, E, y0, A, O);
    const uint32_t U = (M[0] & REC_NTOT) + (M[1] & REC_NTOT) + (M[2] & REC_NTOT) + (M[3] & REC_NTOT);
    bool pois = on && ((M[0] | M[1] | M[2] | M[3]) & REC_POISON);
    bool own = false, spilled = false;
    bool active = on && !pois && A != 0;
    bool counted = true;                      // activity of this (group, gate) not yet counted
    const uint32_t sig = d1.y;
    if (RERUN && on) {
        const uint64_t b = (uint64_t)__ldg(p.prev_idx + grp_gi(G)) * (uint32_t)p.n_gates + (sig - (uint32_t)p.n_pi);
        counted = (__ldg(p.pois_prev + (b >> 5)) >> (b & 31u)) & 1u;
    }
    uint8_t* oreg = grp_row(G) + (size_t)d1.x * GRP_STRIDE(p);
    unsigned long long tb = 0;
    // spill-heap requests of the warp's gates: one bump allocation per warp
    const bool want = active && U < OFF_LIMIT && U > (uint32_t)p.W;
    const uint32_t need = want ? (U + 3u) & ~3u : 0u;
    const uint32_t wm = __ballot_sync(FULL, want);
    unsigned long long wb = 0;
    if (wm) {
        const uint32_t incl = warp_incl_scan(need, lane);
        const uint32_t tot = __shfl_sync(FULL, incl, 31);
        const int lead = __ffs(wm) - 1;
        unsigned long long base = 0;
        if (lane == lead) base = atomicAdd(p.spill_top, (unsigned long long)tot);
        wb = __shfl_sync(FULL, base, lead) + (incl - need);
    }
    if (active) {
        if (U >= OFF_LIMIT) {
            own = true;
        } else if (U <= (uint32_t)p.W) {
            tb = reinterpret_cast<unsigned long long>(oreg + times_off(A));
        } else {
            if (wb + need > p.spill_words) {
                own = true;
            } else {
                tb = reinterpret_cast<unsigned long long>(p.spill + wb);
                __stcg(reinterpret_cast<unsigned long long*>(oreg + REG_SPILLPTR), tb);
                spilled = true;
            }
        }
        if (own) {
            pois = true;
            active = false;
        }
    }
    if (on && !active) {                      // finished here: constant output, or poisoned
        __stcg(grp_rec(G) + (size_t)d1.x * GRP_RSTRIDE(p), make_uint4(y0, 0u, 0u, pois ? REC_POISON : 0u));
        if (pois) {
            if (!RERUN || counted) poison_bit(p, grp_gi(G), sig);
            if (own) p.ovf[grp_gi(G)] = 1;
        }
    }
    const uint32_t bal = __ballot_sync(FULL, active);
    if (active) {
        const uint32_t qe = q_s + 4u * QW * (uint32_t)__popc(bal & lanemask_lt());
        sts_u32x4(qe + 4 * Q_TTK, make_uint4(d1.z, sig, d1.x, y0));
        // the per-gate pass's addresses are formed here, where a lane is a
        // gate (1/32 of the cost of forming them in the pass)
        sts_u32x4(qe + 4 * Q_A, make_uint4(A, (uint32_t)g,
                                           (counted ? QF_COUNT : 0u) | (spilled ? QF_SPILL : 0u) | (d1.w << 8),
                                           (uint32_t)g * 4u * (uint32_t)p.box.nk));
        sts_u64(qe + 4 * Q_TB, tb);
        sts_u32(qe + 4 * Q_AROW, sig * (uint32_t)p.n_vdd + (uint32_t)p.box.k0);
        // the slots of A alike in every input value and observable-event bit
        // (pair-major groups of one pair: the common case): the per-gate pass
        // takes its per-slot bits from this word instead of extracting them
        {
            uint32_t ub = UNI_ALIKE;
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const uint32_t xa = X[q] & A, oa = O[q] & A;
                if ((xa != 0u && xa != A) || (oa != 0u && oa != A)) ub = 0u;
                ub |= (xa ? 1u << q : 0u) | (oa ? 16u << q : 0u);
            }
            sts_u32(qe + 4 * Q_UNI, ub & UNI_ALIKE ? ub : 0u);
        }
        sts_u64(qe + 4 * Q_OREG, reinterpret_cast<unsigned long long>(oreg));
#ifdef AVFS_CHECKS
        AVFS_CHECK(!spilled || wb + need <= p.spill_words);
        sts_u32(qe + 4 * Q_CAP, spilled ? need : ((uint32_t)p.region_bytes - times_off(A)) / 4u);
#endif
        sts_u32x4(qe + 4 * Q_X, make_uint4(X[0], X[1], X[2], X[3]));
        sts_u32x4(qe + 4 * Q_E, make_uint4(O[0], O[1], O[2], O[3]));      // observable events
        sts_u32x4(qe + 4 * Q_AQ, make_uint4(AQ[0], AQ[1], AQ[2], AQ[3]));
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            unsigned long long itb = reinterpret_cast<unsigned long long>(p.zero);
            unsigned long long eb = reinterpret_cast<unsigned long long>(p.pi_ents);
            if ((uint32_t)q < K && (loc[q] & LOC_KIND) != LOC_PI) {
                const uint8_t* r = grp_row(G) + (size_t)(loc[q] & LOC_ID) * GRP_STRIDE(p);
                eb = reinterpret_cast<unsigned long long>(r);
                itb = (M[q] & REC_SPILL) ? __ldcg(reinterpret_cast<const unsigned long long*>(r + REG_SPILLPTR))
                                         : reinterpret_cast<unsigned long long>(r + times_off(AQ[q]));
#if AVFS_PF_L2
                // the observable input's entries and times -> L2 now (one bulk
                // prefetch of its extent, at most 1 KB), so the per-gate
                // pass's dependent loads of them hit L2 (prefetching the
                // pins' delay-table rows as well measured slower: spills)
                if (O[q]) {
                    const uint32_t ne = 4u * (uint32_t)__popc(AQ[q]), nt = 4u * (M[q] & REC_NTOT);
                    if (M[q] & REC_SPILL) {
                        l2_prefetch(r, ne);
                        l2_prefetch(reinterpret_cast<const void*>(itb), nt);
                    } else {
                        l2_prefetch(r, times_off(AQ[q]) + nt);
                    }
                }
#endif
            }
            sts_u64(qe + 4 * Q_ENTB + 8 * q, eb);
            sts_u64(qe + 4 * Q_ITB + 8 * q, itb);
        }
    }
    __syncwarp();                             // queue entries -> the item phase's lanes
    return __popc(bal);
}

// One filter step (readings C3, C4): y is the gate's value after the input
// event at t; a change either cancels the pending last output (it lies after
// t) or pushes t + d.
struct Filt {
    uint32_t proj, cnt;
    float tl;
    __device__ __forceinline__ void step(float t, bool live, uint32_t y, float d, float* out) {
        const float co = t + d;
        const bool change = live && y != proj;
        const bool cancel = change && tl > t;
        const bool push = change && !cancel;
        if (push) __stcg(out + cnt, co);
        cnt = cnt + (push ? 1u : 0u) - (cancel ? 1u : 0u);
        tl = push ? co : (cancel ? -AVFS_INF : tl);
        proj = y;
    }
};

// Merge of at most two sorted lists (pins p0 < p1; list 1 may be empty), the
// next element of each list already loaded (one element of lookahead).
#ifndef AVFS_LOOKAHEAD
#define AVFS_LOOKAHEAD 3
#endif
#ifndef AVFS_MERGE_UNROLL
#define AVFS_MERGE_UNROLL 2        // merge loop unrolled twice: no loop-carried register copies
#endif
constexpr int MERGE_UNROLL = AVFS_MERGE_UNROLL;
#ifndef AVFS_NOREFILL_LOOP
#define AVFS_NOREFILL_LOOP 1
#endif
#ifndef AVFS_UNIFORM_OFF
#define AVFS_UNIFORM_OFF 1
#endif
// The merge loop proper; REFILL = false when every lane's lists fit the
// window (no loads inside the loop).
template <bool REFILL>
__device__ __forceinline__ uint32_t merge_two_loop(float (&w0)[AVFS_LOOKAHEAD], float (&w1)[AVFS_LOOKAHEAD],
                                                   const float* a0, int n0, const float* a1, int n1, uint32_t bits,
                                                   uint32_t tm0, uint32_t tm1, uint32_t proj, uint32_t tt, float4 dl,
                                                   float* out, uint32_t steps) {
    constexpr int D = AVFS_LOOKAHEAD;
    // list positions as 32-bit indices (next element to load) against fixed
    // bases and counts: one address multiply-add per refill, no 64-bit
    // pointer updates
    uint32_t i0 = D, i1 = D;
    Filt F{proj, 0u, -AVFS_INF};
#pragma unroll MERGE_UNROLL
    for (uint32_t it = 0; it < steps; ++it) {
        const bool p = w1[0] < w0[0];                 // ties: the lower pin first (reading C5)
        const float t = fminf(w0[0], w1[0]);
        float nx = AVFS_INF;
        if (REFILL) {
            const uint32_t ix = p ? i1 : i0;
            nx = (int)ix < (p ? n1 : n0) ? ld_f32((p ? a1 : a0) + ix) : AVFS_INF;
            i1 += p ? 1u : 0u;
            i0 += p ? 0u : 1u;
        }
#pragma unroll
        for (int i = 0; i + 1 < D; ++i) {
            w1[i] = p ? w1[i + 1] : w1[i];
            w0[i] = p ? w0[i] : w0[i + 1];
        }
        w1[D - 1] = p ? nx : w1[D - 1];
        w0[D - 1] = p ? w0[D - 1] : nx;
        const bool live = t < AVFS_INF;
        bits ^= live ? (p ? tm1 : tm0) : 0u;
        const uint32_t y = (tt >> bits) & 1u;
        F.step(t, live, y, p ? (y ? dl.w : dl.z) : (y ? dl.y : dl.x), out);
    }
    return F.cnt;
}

__device__ __forceinline__ uint32_t merge_two(const float* a0, int n0, const float* a1, int n1, uint32_t bits,
                                              uint32_t tm0, uint32_t tm1, uint32_t proj, uint32_t tt, float4 dl,
                                              float* out, uint32_t steps) {
    // a window of the next AVFS_LOOKAHEAD elements of each list lives in
    // registers: their loads are issued together up front, and a refill load
    // is consumed AVFS_LOOKAHEAD advances of its list later; when no lane's
    // lists are longer than the window (the common case) the loop has no
    // loads at all
    constexpr int D = AVFS_LOOKAHEAD;
    float w0[D], w1[D];
#pragma unroll
    for (int i = 0; i < D; ++i) {
        w0[i] = n0 > i ? ld_f32(a0 + i) : AVFS_INF;
        w1[i] = n1 > i ? ld_f32(a1 + i) : AVFS_INF;
    }
#if AVFS_NOREFILL_LOOP
    if (__all_sync(FULL, n0 <= D && n1 <= D))
        return merge_two_loop<false>(w0, w1, a0, n0, a1, n1, bits, tm0, tm1, proj, tt, dl, out, steps);
#endif
    return merge_two_loop<true>(w0, w1, a0, n0, a1, n1, bits, tm0, tm1, proj, tt, dl, out, steps);
}

// Delay of arc e = 2 pin + pol of sorted gate `gate` at operating point k,
// evaluated in the sweep (delay_in_sweep: Eq. (4)/(9) as in delay_kernel).
__device__ __noinline__ float sweep_delay(const DelayDesc* __restrict__ dd, const double* __restrict__ coef,
                                          const double* __restrict__ vdd, int n_isl, int deg_v, int deg_c,
                                          double v_min, double v_max, double quantum, int32_t* err, uint32_t gate,
                                          int k, int e) {
    const DelayDesc& D = dd[gate];
    const double v = __ldg(vdd + (size_t)k * n_isl + D.island);
    const double x = (v - v_min) / (v_max - v_min);
    const int nb = (deg_v + 1) * (deg_c + 1);
    bool bad;
    const float d = arc_delay(coef + D.coef_off + e * nb, deg_v, deg_c, x, D.z, D.dnom[e], quantum, bad);
    if (bad) atomicOr(err, 1);
    return d;
}

// Delay of arc e = 2 pin + pol of a queued gate at slot operating point
// k0 + krel: the table entry [gate][pin][krel][pol] (DT), or evaluated here.
template <bool DT>
__device__ __forceinline__ float item_delay(const SweepParams& p, uint32_t gate, int krel, int e) {
    if (DT) return __ldg(p.dtab + (((size_t)gate * 4 + (e >> 1)) * (uint32_t)p.box.nk + krel) * 2 + (e & 1));
    const DelayParams& P = p.dp;
    return sweep_delay(P.dd, P.coef, P.vdd, P.n_isl, P.deg_v, P.deg_c, P.v_min, P.v_max, P.quantum, P.err, gate,
                       p.box.k0 + krel, e);
}

// Merge of up to four sorted lists (list q = pin q, n[q] = 0 if unused);
// delays from the table (or evaluated) per step.
template <bool DT>
__device__ __forceinline__ uint32_t merge_four(const SweepParams& p, const float* const (&a_in)[4], const int (&n_in)[4],
                                               uint32_t bits, uint32_t proj, uint32_t tt, uint32_t gate, int krel,
                                               float* out, uint32_t steps) {
    float h[4];
    const float* a[4];
    int n[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        a[q] = a_in[q];
        n[q] = n_in[q];
        h[q] = n[q] > 0 ? ld_f32(a[q]) : AVFS_INF;
        a[q] += 1;
        n[q] -= 1;
    }
    Filt F{proj, 0u, -AVFS_INF};
#pragma unroll 1
    for (uint32_t it = 0; it < steps; ++it) {
        float t = h[0];
        int pm = 0;
#pragma unroll
        for (int q = 1; q < 4; ++q) {
            const bool lt = h[q] < t;
            t = lt ? h[q] : t;
            pm = lt ? q : pm;
        }
        const float* ap = a[0];
        int np = n[0];
#pragma unroll
        for (int q = 1; q < 4; ++q)
            if (pm == q) { ap = a[q]; np = n[q]; }
        const float nx = np > 0 ? ld_f32(ap) : AVFS_INF;
#pragma unroll
        for (int q = 0; q < 4; ++q)
            if (pm == q) { h[q] = nx; a[q] = ap + 1; n[q] = np - 1; }
        const bool live = t < AVFS_INF;
        bits ^= live ? (1u << pm) : 0u;
        const uint32_t y = (tt >> bits) & 1u;
        F.step(t, live, y, live ? item_delay<DT>(p, gate, krel, 2 * pm + (int)y) : 1.0f, out);
    }
    return F.cnt;
}

// The end of a queued gate's pass: its entries, record, activity per
// (signal, point) (reading C15, counted once per slot group across rerun
// rounds), latest PO arrival.  The queue words are read again here
// rather than held in registers through the merge.
template <bool RERUN>
__device__ __forceinline__ void gate_output(const SweepParams& p, const Grp& G, uint32_t qe, uint32_t n_out,
                                            uint32_t off, bool big, int lane, uint32_t lmask, int krel,
                                            uint32_t& encb) {
    const uint4 w0 = lds_u32x4(qe + 4 * Q_TTK);
    const uint32_t A = lds_u32(qe + 4 * Q_A);
    const bool v = (A >> lane) & 1u;
    if (!v) n_out = 0;
    AVFS_CHECK(!v || big || off + n_out <= lds_u32(qe + 4 * Q_CAP));
    if (v) {
        uint32_t* oent = reinterpret_cast<uint32_t*>(lds_u64(qe + 4 * Q_OREG));
        __stcg(oent + __popc(A & lmask), min(n_out, ENT_N) | (off << ENT_OFF_SHIFT));
        if (n_out && (w0.x & (1u << 24))) {
            const float* o = reinterpret_cast<const float*>(lds_u64(qe + 4 * Q_TB)) + off;
            atomicMax(p.latest + p.box.k0 + krel, __float_as_uint(__ldcg(o + n_out - 1)));
        }
    }
    const uint32_t Eo = __ballot_sync(FULL, n_out != 0u);
    const uint32_t tot = __reduce_add_sync(FULL, n_out);
    const uint32_t fl = lds_u32(qe + 4 * Q_FLAG) | (big ? (QF_POISON | QF_OWN) : 0u);
    const bool pois = fl & QF_POISON, counted = fl & QF_COUNT;
    if (n_out && counted && !pois)
        atomicAdd(p.act + (lds_u32(qe + 4 * Q_AROW) + (uint32_t)krel), (unsigned long long)n_out);
    if (lane == 0) {
        const uint32_t meta = pois ? REC_POISON : (tot | ((fl & QF_SPILL) ? REC_SPILL : 0u));
        __stcg(grp_rec(G) + (size_t)w0.z * GRP_RSTRIDE(p), make_uint4(w0.w, pois ? 0u : Eo, pois ? 0u : A, meta));
        if (pois) {
            if (!RERUN || counted) poison_bit(p, grp_gi(G), w0.y);
            if (fl & QF_OWN) p.ovf[grp_gi(G)] = 1;
        } else {
            encb += (1u + (fl >> 8)) * (uint32_t)__popc(Eo);
        }
    }
}

// Phase B, one queued gate per pass, lane = slot (pair-major groups: a
// gate's observable slots are mostly all 32 operating points of one pair,
// with alike event counts): merge, outputs, entries, activity and the
// gate's record, all in registers.
template <bool RERUN, bool DT>
__device__ __forceinline__ void phase_b(const SweepParams& p, const Grp& G, int nq, uint32_t q_s, int lane) {
    const uint32_t lmask = (1u << lane) - 1u;
    const int krel = G.krel;
    uint32_t encb = 0;                                 // this batch's encoding units (lane 0)
    for (int e = 0; e < nq; ++e) {
        PROF_T0();
        const uint32_t qe = q_s + 4u * QW * (uint32_t)e;
        const uint4 w0 = lds_u32x4(qe + 4 * Q_TTK);      // ttk, sig, out, y0
        const uint32_t A = lds_u32(qe + 4 * Q_A);
        const bool v = (A >> lane) & 1u;
        const uint32_t tt = w0.x & 0xffffu;
        // the slot's input values and its inputs with observable events
        // and the (at most two) first inputs with observable events, p0 < p1
        uint32_t bits, use;
        const uint32_t ub = lds_u32(qe + 4 * Q_UNI);
        if (ub) {                                      // warp-uniform: every slot of A alike (phase A)
            bits = ub & 15u;
            use = v ? (ub >> 4) & 15u : 0u;
        } else {
            const uint4 X = lds_u32x4(qe + 4 * Q_X), Ov = lds_u32x4(qe + 4 * Q_E);
            bits = ((X.x >> lane) & 1u) | (((X.y >> lane) & 1u) << 1) | (((X.z >> lane) & 1u) << 2) |
                   (((X.w >> lane) & 1u) << 3);
            use = ((Ov.x >> lane) & 1u) | (((Ov.y >> lane) & 1u) << 1) | (((Ov.z >> lane) & 1u) << 2) |
                  (((Ov.w >> lane) & 1u) << 3);
        }
        // (taking p0, p1 from phase A as well measured slower: 74.6 vs 71.2 ms)
        const int p0 = use ? __ffs(use) - 1 : 0;
        const uint32_t rest = use & (use - 1u);
        const int p1 = rest ? __ffs(rest) - 1 : p0;
        const bool many = (rest & (rest - 1u)) != 0u;
        // their entries (PIs: the PI entry table, reading C2)
        uint32_t e0 = 0, e1 = 0;
        if (use) {
            const uint32_t* eb = reinterpret_cast<const uint32_t*>(lds_u64(qe + 4 * Q_ENTB + 8 * p0));
            AVFS_CHECK((lds_u32(qe + 4 * Q_AQ + 4 * p0) >> lane) & 1u);
            e0 = __ldcg(eb + __popc(lds_u32(qe + 4 * Q_AQ + 4 * p0) & lmask));
            AVFS_CHECK((e0 & ENT_N) >= 1u);
        }
        if (rest) {
            const uint32_t* eb = reinterpret_cast<const uint32_t*>(lds_u64(qe + 4 * Q_ENTB + 8 * p1));
            AVFS_CHECK((lds_u32(qe + 4 * Q_AQ + 4 * p1) >> lane) & 1u);
            e1 = __ldcg(eb + __popc(lds_u32(qe + 4 * Q_AQ + 4 * p1) & lmask));
            AVFS_CHECK((e1 & ENT_N) >= 1u);
        }
        const uint32_t gate = lds_u32(qe + 4 * Q_GATE);
        float4 dl = make_float4(1.0f, 1.0f, 1.0f, 1.0f);
        if (use && !many) {
            if (DT) {                                  // (fall, rise) of each pin: one 8-B load
                const uint32_t dr = lds_u32(qe + 4 * Q_DROW) + (uint32_t)krel;
                const float2* db = reinterpret_cast<const float2*>(p.dtab);
                const float2 d0 = __ldg(db + (dr + (uint32_t)p0 * (uint32_t)p.box.nk));
                const float2 d1 = __ldg(db + (dr + (uint32_t)p1 * (uint32_t)p.box.nk));
                dl = make_float4(d0.x, d0.y, d1.x, d1.y);
            } else {
                dl.x = item_delay<DT>(p, gate, krel, 2 * p0);
                dl.y = item_delay<DT>(p, gate, krel, 2 * p0 + 1);
                dl.z = item_delay<DT>(p, gate, krel, 2 * p1);
                dl.w = item_delay<DT>(p, gate, krel, 2 * p1 + 1);
            }
        }
        const int n0 = (int)(e0 & ENT_N), n1 = (int)(e1 & ENT_N);
        const float* a0 = reinterpret_cast<const float*>(lds_u64(qe + 4 * Q_ITB + 8 * p0)) + (e0 >> ENT_OFF_SHIFT);
        const float* a1 = reinterpret_cast<const float*>(lds_u64(qe + 4 * Q_ITB + 8 * p1)) + (e1 >> ENT_OFF_SHIFT);
        uint32_t m = (uint32_t)(n0 + n1);
        // rare: three or four inputs with observable events in this slot
        const float* ap[4];
        int nn[4];
        const bool any_many = __any_sync(FULL, many);
        if (any_many) {
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                ap[q] = p.zero;
                nn[q] = 0;
                if (many && ((use >> q) & 1u)) {
                    const uint32_t* eb = reinterpret_cast<const uint32_t*>(lds_u64(qe + 4 * Q_ENTB + 8 * q));
                    const uint32_t w = __ldcg(eb + __popc(lds_u32(qe + 4 * Q_AQ + 4 * q) & lmask));
                    nn[q] = (int)(w & ENT_N);
                    ap[q] = reinterpret_cast<const float*>(lds_u64(qe + 4 * Q_ITB + 8 * q)) + (w >> ENT_OFF_SHIFT);
                }
            }
            if (many) m = (uint32_t)(nn[0] + nn[1] + nn[2] + nn[3]);
        }
        // output offsets: exclusive prefix of the slots' input counts (all
        // slots alike, the common pair-major case: lane x count)
        const uint32_t steps = __reduce_max_sync(FULL, m);
#if AVFS_UNIFORM_OFF
        const uint32_t off = __reduce_min_sync(FULL, m) == steps ? (uint32_t)lane * m : warp_incl_scan(m, lane) - m;
#else
        const uint32_t off = warp_incl_scan(m, lane) - m;
#endif
        const bool big = __any_sync(FULL, v && m > ENT_N);
        PROF_ACC(2);
        float* out = reinterpret_cast<float*>(lds_u64(qe + 4 * Q_TB)) + off;
        const uint32_t y0 = (w0.w >> lane) & 1u;
        uint32_t n_out;
        if (any_many) {
            if (!many) {                               // the other lanes' (at most two) lists
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    ap[q] = (q == p0) ? a0 : ((q == p1 && rest) ? a1 : p.zero);
                    nn[q] = (q == p0) ? n0 : ((q == p1 && rest) ? n1 : 0);
                }
            }
            n_out = merge_four<DT>(p, ap, nn, bits, y0, tt, gate, krel, out, steps);
        } else {
            n_out = merge_two(a0, n0, a1, rest ? n1 : 0, bits, 1u << p0, rest ? 1u << p1 : 0u, y0, tt, dl, out, steps);
        }
        PROF_ACC(3);
        gate_output<RERUN>(p, G, qe, n_out, off, big, lane, lmask, krel, encb);
        PROF_ACC(4);
    }
    if (lane == 0) sts_u64(G.q + WS_OFF, lds_u64(G.q + WS_OFF) + encb);
    __syncwarp();
}


template <bool SPLIT, bool RERUN, bool DT>
__global__ void __launch_bounds__(AVFS_SWEEP_THREADS, AVFS_SWEEP_MINB) sweep_kernel(const SweepParams p) {
    extern __shared__ __align__(16) uint32_t smem_w[];
    // lane and queue address as opaque values: kept in registers instead of
    // being rematerialised (S2R + address arithmetic) in every per-gate pass
    int lane = threadIdx.x & 31;
    asm volatile("" : "+r"(lane));
    const int warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const uint32_t base_s = smem_u32(smem_w);
    uint32_t q_s = base_s + 4u * (uint32_t)(CTA_HDR_WORDS + warp * WARP_SMEM_WORDS);
    asm volatile("" : "+r"(q_s));
    // narrow netlists: the CTA walks GP slot groups at once, nw / GP warps
    // each; few slot groups: S co-resident CTAs (consecutive blocks, grid a
    // multiple of S) share one group, each taking 1/S of every level
    const int GP = SPLIT ? 1 : p.grp_per_cta, wpg = nw / GP, S = SPLIT ? p.split : 1;
    const int sg = warp / wpg, wl = warp % wpg;
    const uint32_t ctr_s = base_s + 8u * (uint32_t)sg;        // this group's level counters
    Grp G;
    G.q = q_s;
    if (lane == 0) sts_u64(q_s + WS_OFF, 0ull);           // encoding units of this warp
    const int64_t u_end = SPLIT ? p.n_sw * S : p.n_sw;
    const int64_t u_step = SPLIT ? (int64_t)gridDim.x : (int64_t)gridDim.x * GP;
    for (int64_t u = SPLIT ? (int64_t)blockIdx.x : (int64_t)blockIdx.x * GP; u < u_end; u += u_step) {
        const int64_t i0 = SPLIT ? u / S : u;
        const int part = SPLIT ? (int)(u % S) : 0;
        const int64_t i = i0 + sg;
        const bool valid = i < p.n_sw;                 // idle warps still meet every level barrier
        group_setup(p, valid ? i : i0, lane, G);
        if (wl == 0 && lane == 0) {
            sts_u32(ctr_s, 0u);
            sts_u32(ctr_s + 4, 0u);
        }
        if (GP == 1 || GP > 15) __syncthreads();
        else asm volatile("bar.sync %0, %1;" ::"r"(1 + sg), "r"(32 * wpg) : "memory");
        for (int L = 0; L < p.depth; ++L) {
            const int ls0 = __ldg(p.level_ptr + L), le0 = __ldg(p.level_ptr + L + 1);
            int ls = ls0, le = le0;
            if (SPLIT) {
                const int P = (le0 - ls0 + S - 1) / S;
                ls = min(le0, ls0 + part * P);
                le = min(le0, ls + P);
            }
            // batches of QN gates are grabbed from a shared counter; the
            // next level's counter is cleared now (its last users finished
            // before the previous barrier)
            const uint32_t cs = ctr_s + 4u * (uint32_t)(L & 1);
            if (wl == 0 && lane == 0) sts_u32(ctr_s + 4u * (uint32_t)((L + 1) & 1), 0u);
            const int nlv = le - ls;
            // levels of at most one round of batches (narrow netlists): one
            // batch per warp, the level split evenly (batch index from the
            // counter); fewer than two rounds: guided batch sizes, a share of
            // the level's remaining gates, so that the warps finish together;
            // wider: full batches and a split last round
            const bool even = nlv <= QN * wpg;
            const int esz = (nlv + wpg - 1) / wpg;
            const bool guided = nlv < 2 * QN * wpg;
            if (valid) {
                while (true) {
                    uint32_t gb = 0;
                    int bsz = QN;
                    if (even) {
                        uint32_t b = 0;
                        if (lane == 0) b = atoms_add(cs, 1u);
                        gb = __shfl_sync(FULL, b, 0) * (uint32_t)esz;
                        bsz = esz;
                    } else if (guided) {
                        // guided batches: a share of what is left, at most QN
                        // gates, so that the level's last batches are small
                        if (lane == 0) {
                            const int rem = nlv - (int)lds_u32(cs);
                            const int bs = max(min(AVFS_MIN_BATCH, QN), min(QN, (rem + 2 * wpg - 1) / (2 * wpg)));
                            gb = atoms_add(cs, (uint32_t)bs) | ((uint32_t)bs << 24);
                        }
                        gb = __shfl_sync(FULL, gb, 0);
                        bsz = (int)(gb >> 24);
                        gb &= 0xFFFFFFu;
                    } else {
#if AVFS_TAIL_SPLIT
                        // wide levels: full batches, except that the last
                        // round (fewer than a batch per warp left) is split
                        // evenly over the group's warps
                        if (lane == 0) {
                            const int rem = nlv - (int)lds_u32(cs);
                            const int bs = rem >= QN * wpg ? QN : max(AVFS_MIN_BATCH, (rem + wpg - 1) / wpg);
                            gb = atoms_add(cs, (uint32_t)bs) | ((uint32_t)bs << 24);
                        }
                        gb = __shfl_sync(FULL, gb, 0);
                        bsz = (int)(gb >> 24);
                        gb &= 0xFFFFFFu;
#else
                        if (lane == 0) gb = atoms_add(cs, QN);
                        gb = __shfl_sync(FULL, gb, 0);
#endif
                    }
                    if ((int)gb >= nlv) break;
                    const int nb = min(bsz, nlv - (int)gb);
                    PROF_T0();
                    const int nq = phase_a<RERUN>(p, G, ls + (int)gb, nb, q_s, lane);
                    PROF_ACC(1);
                    if (nq) phase_b<RERUN, DT>(p, G, nq, q_s, lane);
                    PROF_ACC(5);
                }
            }
            // this level's stores -> the next levels' loads; with several slot
            // groups per CTA each group syncs only its own warps (named barrier)
            PROF_T0();
            if (GP == 1 || GP > 15) __syncthreads();
            else asm volatile("bar.sync %0, %1;" ::"r"(1 + sg), "r"(32 * wpg) : "memory");
            if (SPLIT) {                                // the other parts of this level (L2 counter)
                if (threadIdx.x == 0) {
                    unsigned int* ctr = p.lvl_sync + i;
                    __threadfence();
                    atomicAdd(ctr, 1u);
                    const unsigned int target = (unsigned int)S * (unsigned int)(L + 1);
                    unsigned int vv;
                    while (true) {
                        asm volatile("ld.acquire.gpu.u32 %0, [%1];" : "=r"(vv) : "l"(ctr) : "memory");
                        if (vv >= target) break;
                        __nanosleep(64);
                    }
                    __threadfence();
                }
                __syncthreads();
            }
            PROF_ACC(6);
        }
    }
    if (lane == 0) {
        const unsigned long long enc = lds_u64(q_s + WS_OFF);
        if (enc) atomicAdd(p.enc_units, enc);
    }
}

int debug_phase_cycles(unsigned long long* out, int reset) {
#ifdef AVFS_PROF_PHASES
    if (cudaMemcpyFromSymbol(out, g_phase_cycles, sizeof(unsigned long long) * 16) != cudaSuccess) return -1;
    if (reset) {
        static const unsigned long long z[16] = {};
        cudaMemcpyToSymbol(g_phase_cycles, z, sizeof z);
    }
    return 16;
#else
    (void)out;
    (void)reset;
    return 0;
#endif
}

int sweep_smem_bytes(int warps_per_cta, int) { return 4 * (CTA_HDR_WORDS + warps_per_cta * WARP_SMEM_WORDS); }

// the sweep instantiations: (split group, rerun round, delay table)
template <bool SPLIT, bool RERUN>
static const void* sweep_fn(bool dt) {
    return dt ? reinterpret_cast<const void*>(sweep_kernel<SPLIT, RERUN, true>)
              : reinterpret_cast<const void*>(sweep_kernel<SPLIT, RERUN, false>);
}
static const void* sweep_fn(bool split, bool rerun, bool dt) {
    return split ? (rerun ? sweep_fn<true, true>(dt) : sweep_fn<true, false>(dt))
                 : (rerun ? sweep_fn<false, true>(dt) : sweep_fn<false, false>(dt));
}

cudaError_t sweep_occupancy(int warps_per_cta, int smem, int* blocks_per_sm) {
    // attributes and occupancy are per (device, shape): computed once, not
    // inside every simulate (host time between the stream's events)
    static int c_dev = -1, c_wpc = -1, c_smem = -1, c_bps = 0;
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev == c_dev && warps_per_cta == c_wpc && smem == c_smem) {
        *blocks_per_sm = c_bps;
        return cudaSuccess;
    }
    int m = 1 << 30;
    cudaError_t e = cudaSuccess;
    for (int v = 0; v < 8 && e == cudaSuccess; ++v) {          // split groups need every CTA resident
        const void* f = sweep_fn(v & 1, (v >> 1) & 1, (v >> 2) & 1);
        int b = 0;
        e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, f, warps_per_cta * 32, smem);
        m = b < m ? b : m;
    }
    *blocks_per_sm = m;
    if (e == cudaSuccess) {
        c_dev = dev;
        c_wpc = warps_per_cta;
        c_smem = smem;
        c_bps = m;
    }
    return e;
}

cudaError_t launch_sweep(const SweepParams& p, bool rerun, int grid, int warps_per_cta, cudaStream_t st) {
    const int smem = sweep_smem_bytes(warps_per_cta, p.grp_per_cta);
    SweepParams q = p;
    void* args[] = {&q};
    const void* f = sweep_fn(p.split > 1, rerun, p.dtab != nullptr);
    // the parts of a split slot group wait for each other: a cooperative
    // launch guarantees that every CTA of the grid is resident (or fails)
    if (p.split > 1) return cudaLaunchCooperativeKernel(f, dim3(grid), dim3(warps_per_cta * 32), args, (size_t)smem, st);
    return cudaLaunchKernel(f, dim3(grid), dim3(warps_per_cta * 32), args, (size_t)smem, st);
}

// ---------------------------------------------------------------------------
// Delay computation kernel (P:L139, P:L152-L160 steps 3-5): one thread per
// (operating point, gate, pin, polarity); fills the table the sweep reads,
// or (dtab null) only checks every delay for d' > 0 (reading C14).
__global__ void delay_kernel(const DelayParams p) {
    // table [gate][pin][k - kv_lo][pol], operating points kv_lo .. kv_hi-1
    // only (the ones the slot range covers): a warp of the sweep's items
    // (consecutive points of one gate) reads a pin's (fall, rise) pairs as
    // one contiguous 8-B-per-lane load
    const int nk = p.kv_hi - p.kv_lo;
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)p.n_gates * 8 * nk) return;
    const int pol = (int)(t & 1);
    const int64_t r = t >> 1;
    const int kv = p.kv_lo + (int)(r % nk);
    const int64_t gp = r / nk;
    const int e = 2 * (int)(gp & 3) + pol;
    const int g = (int)(gp >> 2);
    const DelayDesc& D = p.dd[g];
    float out = 1.0f;
    if (e < 2 * (int)D.k) {
        const double v = p.vdd[(size_t)kv * p.n_isl + D.island];           // gate's island supply (NEXT-2)
        const double x = (v - p.v_min) / (p.v_max - p.v_min);                // phi_V
        const int nb = (p.deg_v + 1) * (p.deg_c + 1);
        bool bad;
        out = arc_delay(p.coef + D.coef_off + e * nb, p.deg_v, p.deg_c, x, D.z, D.dnom[e], p.quantum, bad);
        if (bad) atomicOr(p.err, 1);
    }
    if (p.dtab) p.dtab[t] = out;
}

cudaError_t launch_delays(const DelayParams& p, cudaStream_t st) {
    const int64_t n = (int64_t)(p.kv_hi - p.kv_lo) * p.n_gates * 8;
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

// H4 for the sweep: stimulus words per slot group of the box, bit l of
// p1g[i][sw] = PI i of lane l's pair (0 outside the box).  One warp per
// (word b, group sw): 32 ballots transpose a 32x32 bit block.
__global__ void expand_groups_kernel(const uint32_t* __restrict__ p1, const uint32_t* __restrict__ p2, int32_t words,
                                     int32_t n_pi, const SlotBox box, int64_t n_grp, uint32_t* __restrict__ p1g,
                                     uint32_t* __restrict__ p2g) {
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (gw >= (int64_t)words * n_grp) return;
    const int b = (int)(gw / n_grp);
    const int64_t sw = gw % n_grp;
    const int64_t i = sw * 32 + lane;
    const bool in = i < box.nj * box.nk;
    int64_t pair = box.j0 + (in ? i / box.nk : 0);
    if (pair >= box.n_pairs) pair -= box.n_pairs;
    const uint32_t w1 = in ? p1[pair * words + b] : 0u;
    const uint32_t w2 = in ? p2[pair * words + b] : 0u;
    uint32_t m1 = 0, m2 = 0;
#pragma unroll 4
    for (int bit = 0; bit < 32; ++bit) {
        const uint32_t r1 = __ballot_sync(0xffffffffu, (w1 >> bit) & 1u);
        const uint32_t r2 = __ballot_sync(0xffffffffu, (w2 >> bit) & 1u);
        if (lane == bit) { m1 = r1; m2 = r2; }
    }
    const int pi = b * 32 + lane;
    if (pi < n_pi) {
#if AVFS_PI_GMAJOR
        reinterpret_cast<uint2*>(p1g)[sw * n_pi + pi] = make_uint2(m1, m2);
        (void)p2g;
#else
        p1g[(int64_t)pi * n_grp + sw] = m1;
        p2g[(int64_t)pi * n_grp + sw] = m2;
#endif
    }
}

cudaError_t launch_expand_groups(const uint32_t* p1, const uint32_t* p2, int32_t words, int32_t n_pi,
                                 const SlotBox& box, int64_t n_grp, uint32_t* p1g, uint32_t* p2g, cudaStream_t st) {
    const int64_t threads = (int64_t)words * n_grp * 32;
    const int bs = 256;
    const int64_t grid = (threads + bs - 1) / bs;
    if (grid == 0) return cudaSuccess;
    expand_groups_kernel<<<(unsigned)grid, bs, 0, st>>>(p1, p2, words, n_pi, box, n_grp, p1g, p2g);
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

// H8 for primary inputs: act[pi][k] = number of simulated pairs with p1 != p2
// (pairs of the public range at point k, within the box's pairs).
__global__ void pi_activity_kernel(const uint32_t* __restrict__ p1t, const uint32_t* __restrict__ p2t,
                                   int32_t n_pi, int32_t n_pw, const SlotBox box, int32_t n_vdd,
                                   unsigned long long* act) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n_pi * n_vdd) return;
    const int pi = (int)(t / n_vdd);
    const int k = (int)(t % n_vdd);
    const int64_t P = box.n_pairs;
    int64_t lo = box.slot_first - (int64_t)k * P, hi = box.slot_end - (int64_t)k * P;
    lo = lo < 0 ? 0 : lo;
    hi = hi > P ? P : hi;
    if (box.j0 + box.nj <= P) {                  // a plain pair interval (not wrapped)
        lo = lo > box.j0 ? lo : box.j0;
        hi = hi < box.j0 + box.nj ? hi : box.j0 + box.nj;
    }
    if (k < box.k0 || k >= box.k0 + box.nk) hi = lo;
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
                               const SlotBox& box, int32_t n_vdd, unsigned long long* act, cudaStream_t st) {
    const int64_t n = (int64_t)n_pi * n_vdd;
    if (n == 0) return cudaSuccess;
    pi_activity_kernel<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(p1t, p2t, n_pi, n_pw, box, n_vdd, act);
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

// Slot l of a stored waveform (record + region layout, avfs_internal.h):
// initial value, count and its times; false if the waveform is poisoned.
__device__ __forceinline__ bool read_slot(const GatherRound& R, uint32_t buf, int64_t idx, int l, uint32_t& init,
                                          int& n, const float*& ev) {
#if AVFS_REC_GROUP_MAJOR
    const uint4 rec = R.recs[(size_t)idx * R.n_buf + buf];
#else
    const uint4 rec = R.recs[(size_t)buf * R.n_sw + idx];
#endif
    if (rec.w & REC_POISON) return false;
#if AVFS_REG_GROUP_MAJOR
    const uint8_t* reg = R.pinned + ((int64_t)idx * R.n_buf + buf) * R.region_bytes;
#else
    const uint8_t* reg = R.pinned + ((int64_t)buf * R.n_sw + idx) * R.region_bytes;
#endif
    init = (rec.x >> l) & 1u;
    n = 0;
    ev = nullptr;
    if ((rec.z >> l) & 1u) {
        const uint32_t w = reinterpret_cast<const uint32_t*>(reg)[__popc(rec.z & ((1u << l) - 1u))];
        n = (int)(w & ENT_N);
        const float* tb = (rec.w & REC_SPILL) ? *reinterpret_cast<const float* const*>(reg + REG_SPILLPTR)
                                              : reinterpret_cast<const float*>(reg + times_off(rec.z));
        ev = tb + (w >> ENT_OFF_SHIFT);
    }
    return true;
}

// H9: readback of kept waveforms (PIs from the stimuli, gates from the round
// that holds each slot group's final data).  One thread per (signal, slot).
__global__ void gather_kernel(const GatherParams p) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)p.n_sig * p.n_slots) return;
    const int q = (int)(t / p.n_slots);
    const int64_t s = p.slot0 + t % p.n_slots;
    const int64_t k = s / p.box.n_pairs, j = s % p.box.n_pairs;
    const int64_t pw = j / 32;
    const int64_t jr = j >= p.box.j0 ? j - p.box.j0 : j - p.box.j0 + p.box.n_pairs;
    const int64_t i = jr * p.box.nk + (k - p.box.k0);                  // position in the box (SlotBox)
    const int64_t sw = i >> 5;
    const int lane = (int)(i & 31);
    const uint32_t loc = p.sig_loc[q];
    uint32_t init = 0;
    int n = 0;
    float* tout = p.times ? p.times + t * p.cap : nullptr;
    if ((loc & LOC_KIND) == LOC_PI) {
        const uint32_t w1 = p.p1t[(int64_t)(loc & LOC_ID) * p.n_pw + pw];
        const uint32_t w2 = p.p2t[(int64_t)(loc & LOC_ID) * p.n_pw + pw];
        init = (w1 >> (j & 31)) & 1u;
        n = (int)(((w1 ^ w2) >> (j & 31)) & 1u);
        if (tout) for (int i = 0; i < p.cap; ++i) tout[i] = 0.0f;
    } else {
        const int r = p.sw_round[sw];
        if (r < 0) { atomicOr(p.bad, 1); return; }
        const float* ev;
        if (!read_slot(p.rounds[r], loc & LOC_ID, p.sw_index[sw], lane, init, n, ev)) { atomicOr(p.bad, 2); return; }
        if (tout) for (int i = 0; i < p.cap; ++i) tout[i] = i < n ? __ldcg(ev + i) : 0.0f;
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
    int64_t j;
    int kv;
    const bool valid = box_slot(p.box, sw, lane, j, kv);
    const int64_t pw = j / 32;
    const float T = p.t_clk[kv];
    const uint32_t loc = p.po_loc[o];
    uint32_t init = 0, n = 0, c = 0;
    float last = 0.0f;
    if ((loc & LOC_KIND) == LOC_PI) {
        const uint32_t w1 = p.p1t[(int64_t)(loc & LOC_ID) * p.n_pw + pw];
        const uint32_t w2 = p.p2t[(int64_t)(loc & LOC_ID) * p.n_pw + pw];
        init = (w1 >> (j & 31)) & 1u;
        n = ((w1 ^ w2) >> (j & 31)) & 1u;
        c = (n && 0.0f <= T) ? 1u : 0u;
    } else {
        const int r = p.sw_round[sw];
        const float* ev;
        int nn = 0;
        if (r >= 0 && read_slot(p.rounds[r], loc & LOC_ID, p.sw_index[sw], lane, init, nn, ev)) {
            n = (uint32_t)nn;
            if (valid)
                for (uint32_t e = 0; e < n; ++e) {
                    const float t = __ldcg(ev + e);
                    last = t;
                    c += (t <= T) ? 1u : 0u;
                }
        }
    }
    const bool fail = valid && (((init ^ c) & 1u) != ((init ^ n) & 1u));
    if (fail) atomicAdd(p.fail_po + (int64_t)o * p.n_vdd + kv, 1u);
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
    int64_t j;
    int kv;
    if (!box_slot(p.box, sw, lane, j, kv)) return;
    const int64_t pub = (int64_t)kv * p.box.n_pairs + j;
    const uint32_t f = p.slot_fail[t];
    if (f) atomicAdd(p.fail_pairs + kv, 1u);
    if (p.fail_bits)
        p.fail_bits[p.fb_pairs ? (int64_t)(kv - p.box.k0) * p.box.nj + (j - p.box.j0) : pub - p.box.slot_first] = (uint8_t)f;
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
