// avfs_internal.h -- structures shared by the host runtime (avfs_host.cpp)
// and the sm_100a kernels (avfs_kernels.cu).  Not part of the C-ABI.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace avfs {

// sweep CTA shape (compile-time; A/B knobs via -D)
#ifndef AVFS_SWEEP_THREADS
#define AVFS_SWEEP_THREADS 1024
#endif
#ifndef AVFS_SWEEP_MINB
#define AVFS_SWEEP_MINB (AVFS_SWEEP_THREADS > 768 ? 1 : (AVFS_SWEEP_THREADS > 512 ? 2 : 3))
#endif

#ifndef AVFS_PI_GMAJOR
#define AVFS_PI_GMAJOR 1
#endif

constexpr int KMAX = 4;            // max cell inputs (truth table is 16 bits)
constexpr int MAX_DEG = 7;         // max polynomial degree per variable

// Location code of a waveform: kind in bits 30..31.
constexpr uint32_t LOC_PI = 0u << 30;        // low bits: PI index (waveform derived from stimuli)
constexpr uint32_t LOC_SCRATCH = 1u << 30;   // low bits: scratch buffer id (liveness-coloured)
constexpr uint32_t LOC_PINNED = 2u << 30;    // low bits: pinned id (PO / probe / keep_all)
constexpr uint32_t LOC_KIND = 3u << 30;
constexpr uint32_t LOC_ID = ~LOC_KIND;

// Waveform of one (signal, 32-slot group) (reading C1), in two parts:
//
//  record  uint4 {init, E, A, meta} in the round's record array
//          [group][buffer]: init = bit l is slot l's value before t = 0,
//          E = slots with >= 1 transition, A = slots that own an entry
//          (E is a subset of A), meta = total stored transitions (REC_NTOT)
//          plus REC_POISON / REC_SPILL.  PIs have no record: it is the
//          stimulus words (init = p1, E = A = p1 xor p2, one event at t = 0).
//  region  in the round's arena [group][buffer]: popc(A) entry words, compact
//          in the order of A's set bits (entry = n | off << ENT_OFF_SHIFT: the
//          slot's count and the word offset of its first time), then the
//          binary32 times from byte 128 (times_off: the line after 32
//          entries; regions are line-aligned), so a gate's output is one
//          extent; when the record says REC_SPILL
//          the times live in the spill heap at the 64-bit address stored at
//          byte REG_SPILLPTR.  Regions hold up to W times.
constexpr uint32_t REC_NTOT = 0x0FFFFFFFu;
constexpr uint32_t REC_POISON = 1u << 29;    // events not stored here or upstream (overflow)
constexpr uint32_t REC_SPILL = 1u << 30;
constexpr uint32_t ENT_N = 0xFFFu;           // per-slot count limit 4095
constexpr int ENT_OFF_SHIFT = 12;            // 20-bit time offset: <= 2^20 - 1 times per (signal, group)
constexpr uint32_t OFF_LIMIT = 1u << 20;
constexpr int REG_SPILLPTR = 128;
constexpr int REG_TIMES = 144;

// Gate descriptor, 32 B, read by one lane per gate (P:L154 step 1).
struct alignas(16) GateDesc {
    uint32_t in_loc[KMAX];   // location codes of the inputs (LOC_PI | pi, or kind | buffer id)
    uint32_t out_loc;        // arena buffer id of the output
    uint32_t sig;            // output signal id (activity row)
    uint32_t ttk;            // bits 0..15 truth table, 16..23 #inputs, 24..31 flags (bit 24: PO)
    uint32_t fanout;         // reading pins of the output (algorithmic-byte accounting)
};
static_assert(sizeof(GateDesc) == 32, "GateDesc layout");

// Inputs of the delay computation: per sorted gate.  The delay of
// arc (pin, pol) at supply v is Eq. (4)/(9) with the cell's coefficients
// beta[deg_v+1][deg_c+1] (block at coef_off + (2 pin + pol) nb, nb =
// (deg_v+1)(deg_c+1)), x = phi_V(v) and the gate's z = phi_C(c_load)
// (computed at load from the gate's load, 0 when deg_c = 0).
struct alignas(16) DelayDesc {
    double dnom[2 * KMAX];   // [pin][pol] nominal delay, ps
    double z;                // phi_C(c_g)
    uint32_t coef_off;       // offset (doubles) of the cell's [pin][pol][deg_v+1][deg_c+1] block
    uint32_t k;
    uint32_t island;         // voltage island (NEXT-2)
    uint32_t pad[3];
};
static_assert(sizeof(DelayDesc) == 96, "DelayDesc layout");

// The slots of a simulate.  Public slot s = k * n_pairs + j (stimulus pair j,
// operating point k); the simulated range [slot_first, slot_end) lies in the
// box pairs j0, j0 + 1, ... (nj of them, modulo n_pairs: a range that
// straddles two rows starts at its first pair and wraps around) x points
// [k0, k0 + nk).  Internally the box is enumerated pair-major,
// i = ((j - j0) mod n_pairs) * nk + (k - k0), so that a pair's
// operating points are adjacent: slot group sw = i / 32, lane i % 32.  A
// group's slots then share (mostly) one input pair and differ only in Vdd --
// the same transitions, scaled in time -- so their event counts are alike.
struct SlotBox {
    int64_t n_pairs;
    int64_t j0, nj;
    int32_t k0, nk;
    int64_t slot_first, slot_end;
};

struct DelayParams {
    const DelayDesc* __restrict__ dd;
    int32_t n_gates;
    const double* __restrict__ coef;         // [cell][pin][pol][deg_v+1][deg_c+1]
    int32_t deg_v, deg_c;
    const double* __restrict__ vdd;          // [n_vdd][n_isl] volts
    int32_t n_vdd;
    int32_t n_isl;
    int32_t kv_lo, kv_hi;                    // operating points with simulated slots (the box's k0, k0 + nk)
    double v_min, v_max;
    double quantum;                          // 0: F mode
    float* dtab;                             // [n_gates][pin 4][kv_hi - kv_lo][pol 2] delays (binary32), ps; null: check only
    int32_t* err;                            // bit 0: non-positive delay
};

struct SweepParams {
    const GateDesc* __restrict__ gates;     // sorted by level
    const int32_t* __restrict__ level_ptr;  // [depth+1] offsets into gates (level 1..depth)
    int32_t depth;
    int32_t n_gates;
    const float* __restrict__ dtab;         // [n_gates][4][box.nk][2] delays, or null: evaluated in the sweep
    DelayParams dp;                         // delay model (used when dtab is null)
    // stimulus words per slot group (bit l: lane l's pair): uint2 {p1, p2}
    // [n_grp][n_pi] (AVFS_PI_GMAJOR), else p1g / p2g [n_pi][n_grp]
    const uint32_t* __restrict__ p1g;
    const uint32_t* __restrict__ p2g;
    int64_t n_grp;                          // slot groups of the box
    SlotBox box;
    int32_t n_vdd;
    // slot groups of this run: sw = sw_list ? sw_list[i] : sw_first + i, i < n_sw
    const int32_t* __restrict__ sw_list;
    int64_t sw_first;
    int64_t n_sw;                           // slot groups in this launch
    int64_t i_base;                         // index of this launch's first group within the round
    int64_t pin_n_sw;                       // slot groups in the round (arena / records / ovf flags)
    // arena of the round: [buffer][pin_n_sw][region]; buffers = kept signals, then scratch
    uint8_t* arena;
    int64_t region_bytes;
    uint4* recs;                            // [buffer][pin_n_sw] records (or [pin_n_sw][n_buf])
    int64_t n_buf;                          // arena buffers (kept + scratch)
    int32_t W;                              // in-place time capacity per region (words)
    int32_t grp_per_cta;                    // slot groups a sweep CTA walks at once (power of 2)
    int32_t split;                          // sweep CTAs sharing one slot group (grp_per_cta == 1)
    unsigned int* lvl_sync;                 // [n_sw] level counters of split groups (zeroed per round)
    int32_t n_pi;                           // gate index = output signal - n_pi
    // spill heap of the round: gates whose inputs carry more than W events
    // store their times here (bump allocation in words, 16-B granules)
    float* spill;
    unsigned long long* spill_top;          // words handed out (counts failed requests too)
    uint64_t spill_words;                   // heap capacity
    // poison bitmaps [group index in round][n_gates] bits: this round's, and
    // the previous round's (null on pass 0): set = poisoned and not counted yet
    uint32_t* pois;
    const uint32_t* pois_prev;
    const int32_t* prev_idx;                // [n_sw] group's index in the previous round
    const float* zero;                      // 4 words of 0.0f: the time of every PI event (reading C2)
    const uint32_t* pi_ents;                // 32 entries {n = 1, offset 0}: every PI slot with an event
    // outputs
    unsigned long long* act;                // [n_signals][n_vdd]
    unsigned int* latest;                   // [n_vdd] float bits (non-negative)
    int32_t* ovf;                           // [n_sw] overflow flag per slot group
    unsigned long long* enc_units;          // sum over gates of (1 + fanout) * #slots with events
};

// launch wrappers (avfs_kernels.cu)
int sweep_smem_bytes(int warps_per_cta, int grp_per_cta);
int debug_phase_cycles(unsigned long long* out, int reset);   // -DAVFS_PROF_PHASES builds only
cudaError_t sweep_occupancy(int warps_per_cta, int smem, int* blocks_per_sm);
cudaError_t launch_delays(const DelayParams& p, cudaStream_t st);
cudaError_t launch_sweep(const SweepParams& p, bool rerun, int grid, int warps_per_cta, cudaStream_t st);
cudaError_t launch_expand(const uint32_t* p1, const uint32_t* p2, int64_t n_pairs, int32_t words,
                          int32_t n_pi, int32_t n_pw, uint32_t* p1t, uint32_t* p2t, cudaStream_t st);
cudaError_t launch_expand_groups(const uint32_t* p1, const uint32_t* p2, int32_t words, int32_t n_pi,
                                 const SlotBox& box, int64_t n_grp, uint32_t* p1g, uint32_t* p2g, cudaStream_t st);
cudaError_t launch_pi_activity(const uint32_t* p1t, const uint32_t* p2t, int32_t n_pi, int32_t n_pw,
                               const SlotBox& box, int32_t n_vdd, unsigned long long* act, cudaStream_t st);
cudaError_t launch_compact_overflow(const int32_t* ovf, int64_t n_sw, const int32_t* sw_list,
                                    int64_t sw_first, int32_t* out_list, int32_t* out_prev,
                                    int32_t* out_count, cudaStream_t st);

struct GatherRound {       // one simulated round for readback
    const uint8_t* pinned;      // arena (kept buffers first)
    const uint4* recs;          // records [buffer][n_sw] (or [n_sw][n_buf])
    int64_t region_bytes;
    int64_t n_sw;
    int64_t n_buf;
};
struct GatherParams {
    const uint32_t* sig_loc;    // [n_sig] location codes (LOC_PI | pi, or LOC_PINNED | arena buffer)
    int32_t n_sig;
    int64_t slot0, n_slots;
    SlotBox box;
    int32_t n_pw;
    const uint32_t* p1t;        // [n_pi][n_pw] pair-warp stimulus words (PI waveforms)
    const uint32_t* p2t;
    const int32_t* sw_round;    // [n_grp] round index holding the final data (-1: not simulated)
    const int32_t* sw_index;    // [n_grp] index within that round
    GatherRound rounds[8];
    int32_t cap;
    uint8_t* init;
    int32_t* count;
    float* times;
    int32_t* bad;               // set when a requested slot was not simulated / still poisoned
};
cudaError_t launch_gather(const GatherParams& p, cudaStream_t st);

// NEXT-1 capture analysis over the kept PO waveforms
struct CaptureParams {
    const uint32_t* po_loc;     // [n_po] LOC_PI | pi, or LOC_PINNED | arena buffer
    int32_t n_po;
    int32_t n_vdd;
    const float* t_clk;         // [n_vdd]
    int64_t sw_lo, n_sw;        // simulated slot groups [sw_lo, sw_lo + n_sw)
    SlotBox box;
    int32_t n_pw;
    const uint32_t* p1t;
    const uint32_t* p2t;
    const int32_t* sw_round;
    const int32_t* sw_index;
    GatherRound rounds[8];
    uint32_t* slot_fail;        // [n_sw * 32]
    uint32_t* slot_last;        // [n_sw * 32] float bits
    uint32_t* fail_po;          // [n_po][n_vdd]
    uint32_t* fail_pairs;       // [n_vdd]
    uint32_t* hist;             // [n_vdd][n_bins] or null
    int32_t n_bins;
    float lo, width;
    uint8_t* fail_bits;         // [simulated slots] in public slot order, or null
    int32_t fb_pairs;           // pair range: fail_bits[(k - k0) * nj + j - j0], else [slot - slot_first]
};
cudaError_t launch_capture(const CaptureParams& p, cudaStream_t st);

// NEXT-4 switching energy: out[k] += 1/2 sum_g act[n_pi+g][k] c[g] v_k^2
cudaError_t launch_energy(const unsigned long long* act, const double* c_load, const double* vdd,
                          const int32_t* island, int32_t n_isl, int32_t n_pi, int32_t n_gates, int32_t n_vdd,
                          double* out, cudaStream_t st);

}  // namespace avfs
