/*
 * avfs.h -- C-ABI of libavfs: B200-native (sm_100a) waveform-accurate logic
 * time simulation under many supply-voltage operating points.
 *
 * The calls follow the paper's statement of the problem (Schneider &
 * Wunderlich, DATE'20; /root/reference/PAPER.md cited "P:L<n>"):
 *   (1) netlist + timing            P:L141 step 1, P:L148 (pin-to-pin delays
 *                                   with output polarity, inertial = propagation)
 *   (1') cell library + coefficients P:L133, P:L139 (per cell / pin / polarity
 *                                   polynomial, Eq. 4, evaluated in FP64)
 *   (2) operating points            P:L141 step 2, P:L152 (parameter memory)
 *   (3) stimuli + simulate          P:L141 step 3, P:L164-L175 (3-D parallel:
 *                                   gates x stimuli x operating points)
 *   (4) waveform analysis           P:L141 step 4 (responses, switching
 *                                   activity, transition times)
 *
 * Conventions
 *   signals : primary inputs are 0..n_pi-1; gate g drives signal n_pi+g.
 *   polarity: pol 0 = output falls, pol 1 = output rises.
 *   slots   : one (stimulus pair j, operating point k); public slot index
 *             s = k * n_pairs + j (Vdd-major, reading C16).
 *   times   : picoseconds, binary32 on the device; delays are evaluated in
 *             binary64 and rounded once to binary32 (reading C11).
 *   truth table: bit b of truth_table is the cell output for the input
 *             vector b, pin 0 = least significant bit.  At most 4 inputs.
 *
 * Ownership: every input array is copied; the caller keeps ownership.
 * Outputs go to caller-allocated buffers.  The context owns all device
 * memory.  No call retains a caller pointer after it returns.
 *
 * Errors: every call returns an avfs_status; avfs_last_error() gives text
 * (owned by the context, valid until the next call on it).  No exception
 * crosses the ABI.  AVFS_ERR_CUDA is sticky: destroy the context.
 * State order: library -> netlist -> {stimuli, operating points, options,
 * slot range} -> simulate -> get_*.  Out-of-order calls: AVFS_ERR_STATE.
 * A context is not thread-safe; use one per thread / device.
 */
#ifndef AVFS_H
#define AVFS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct avfs_ctx avfs_ctx;

typedef enum {
    AVFS_OK = 0,
    AVFS_ERR_ARG = 1,           /* bad argument (null, range, arity, size)     */
    AVFS_ERR_PARSE = 2,         /* .bench text or netlist structure (cycle)     */
    AVFS_ERR_STATE = 3,         /* call out of order / host-only context        */
    AVFS_ERR_CUDA = 4,          /* CUDA runtime error (sticky)                  */
    AVFS_ERR_NOMEM = 5,         /* device or host allocation failed             */
    AVFS_ERR_DELAY_NONPOS = 6,  /* some d' = d_nom (1 + f(P)) <= 0 (reading C14) */
    AVFS_ERR_CAPACITY = 7       /* waveform capacity still exceeded after the
                                   allowed rerun rounds (reading C17)          */
} avfs_status;

/* Create a context on CUDA device `cuda_device`.  cuda_device = -1 creates a
 * host-only context: library/netlist loading and inspection work, simulate
 * and get_* return AVFS_ERR_STATE (used by CPU-only tests). */
avfs_status avfs_create(int cuda_device, avfs_ctx **out);
void avfs_destroy(avfs_ctx *ctx);
const char *avfs_last_error(const avfs_ctx *ctx);
const char *avfs_status_string(avfs_status st);
/* "avfs <version> sm_100a" */
const char *avfs_version(void);

/* ---------------------------------------------------------------- (1') */
typedef struct {
    const char *name;      /* e.g. "NAND2"; used by avfs_load_bench        */
    int32_t n_inputs;      /* 1..4                                          */
    uint16_t truth_table;  /* bit b = output for input vector b             */
} avfs_cell;

/* Cell library with Eq. (4) coefficients:
 *   beta[cell][pin<4][pol<2][deg_v+1][deg_c+1], row-major (reading C9),
 *   beta[..][i][j] multiplies phi_V(v)^i * phi_C(c)^j with
 *   phi_V(v) = (v - v_min)/(v_max - v_min),
 *   phi_C(c) = (log2 c - log2 c_min)/(log2 c_max - log2 c_min).
 * f(P) approximates d/d_nom - 1 (Eq. 3); the delay is d' = d_nom (1 + f)
 * (Eq. 9).  0 <= deg_v, deg_c <= 7.  Pins >= n_inputs are ignored.
 * Loading a library invalidates a loaded netlist.                       */
avfs_status avfs_load_library(avfs_ctx *ctx, int32_t n_cells, const avfs_cell *cells,
                              int32_t deg_v, int32_t deg_c, const double *beta,
                              double v_min, double v_max, double c_min_fF, double c_max_fF);

/* ---------------------------------------------------------------- (1) */
/* Combinational netlist (full scan already cut).
 *   gate_cell[n_gates]       cell index into the library
 *   fanin_ptr[n_gates+1]     CSR offsets into fanin_sig (int64)
 *   fanin_sig[E]             driving signal of each input pin, pin order
 *   d_nom_ps[E][2]           nominal pin-to-pin delay per fan-in edge and
 *                            output polarity (SDF stand-in), > 0
 *   c_load_fF[n_gates]       output load per gate; may be NULL iff deg_c == 0
 *   po_sig[n_po]             primary (or pseudo-primary) output signals
 * Gates may be in any order; the library levelises.  Errors:
 * AVFS_ERR_ARG (arity, index, delay <= 0), AVFS_ERR_PARSE (cycle).      */
avfs_status avfs_load_netlist(avfs_ctx *ctx, int32_t n_pi, int32_t n_gates,
                              const int32_t *gate_cell, const int64_t *fanin_ptr,
                              const int32_t *fanin_sig, const double *d_nom_ps,
                              const double *c_load_fF, int32_t n_po, const int32_t *po_sig);

/* ISCAS .bench text: INPUT(x), OUTPUT(x), x = TYPE(a, b, ...), '#' comments.
 * DFF(d) is cut for full scan: its Q becomes a pseudo primary input
 * (numbered after the INPUTs), its D a pseudo primary output.  TYPE with k
 * inputs maps to library cell "TYPEk" (e.g. NAND -> NAND2) or, for k == 1,
 * NOT -> "INV", BUFF/BUF -> "BUF".  Gates are numbered in order of
 * appearance; d_nom_ps is [edge][2] in that order (fan-ins as listed).  */
avfs_status avfs_load_bench(avfs_ctx *ctx, const char *text, size_t len,
                            const double *d_nom_ps, const double *c_load_fF);
/* Signal id of a .bench net name (after avfs_load_bench). */
avfs_status avfs_find_signal(avfs_ctx *ctx, const char *name, int32_t *sig);

typedef struct {
    int32_t n_pi, n_gates, n_po, depth;       /* depth = number of gate levels  */
    int32_t max_fanin, n_scratch_buffers;     /* liveness-coloured buffers      */
    int32_t n_pinned;                         /* POs + probes (or all gates)    */
    int32_t n_dangling;                       /* gate outputs with no reader, not PO */
    int64_t n_edges;
} avfs_netlist_info;
avfs_status avfs_get_netlist_info(avfs_ctx *ctx, avfs_netlist_info *info);
/* level[n_pi + n_gates]: 0 for PIs, 1 + max fan-in level for gates.      */
avfs_status avfs_get_levels(avfs_ctx *ctx, int32_t *level);
/* loc[n_pi + n_gates]: -1 for PIs, scratch buffer id (>= 0) or
 * -2 - pinned id for pinned signals.  Valid after options are set.       */
avfs_status avfs_get_buffer_map(avfs_ctx *ctx, int32_t *loc);

/* ---------------------------------------------------------------- (2) */
/* Operating points: n_vdd supply voltages in volts.             */
avfs_status avfs_set_operating_points(avfs_ctx *ctx, int32_t n_vdd, const double *vdd_volts);

/* NEXT-2 -- per-gate operating points (voltage islands; "gate- and circuit
 * parameters P").  island_of_gate[n_gates] in [0, n_islands) (NULL:
 * all 0); vdd_volts[n_points][n_islands]: operating point k supplies island i
 * with vdd_volts[k][i].  Gate g's delays at point k use vdd[k][island[g]].
 * avfs_set_operating_points(n, v) is the 1-island special case.  Call after
 * the netlist is loaded (loading a netlist resets to one island).        */
avfs_status avfs_set_voltage_islands(avfs_ctx *ctx, int32_t n_islands, const int32_t *island_of_gate,
                                     int32_t n_points, const double *vdd_volts);

/* ---------------------------------------------------------------- (3) */
/* Two-pattern stimuli: p1, p2 are uint32 [n_pairs][ceil(n_pi/32)], bit
 * (i % 32) of word (i / 32) is PI i.  All PIs with p1 != p2 switch at
 * t = 0 (reading C2).  is_device = 0: host pointers, copied before the
 * call returns; 1: device pointers (copied device-to-device before return). */
avfs_status avfs_set_stimuli(avfs_ctx *ctx, int64_t n_pairs, const uint32_t *p1,
                             const uint32_t *p2, int32_t is_device);

/* Restrict simulation to public slots [first_slot, first_slot + n_slots)
 * (multi-GPU sharding).  Default / n_slots < 0: all slots.        */
avfs_status avfs_set_slot_range(avfs_ctx *ctx, int64_t first_slot, int64_t n_slots);

/* Restrict simulation to stimulus pairs [first_pair, first_pair + n_pairs)
 * at every operating point (multi-GPU sharding by pairs: each
 * (pattern, Vdd) is independent).  The slot groups then hold whole pairs'
 * operating-point sweeps, the layout the sweep is fastest on.  Replaces a
 * slot range (and avfs_set_slot_range replaces this); readback accepts the
 * public slots of these pairs.  AVFS_ERR_ARG if n_pairs < 1; at simulate,
 * if the range exceeds the stimulus pairs.                                 */
avfs_status avfs_set_pair_range(avfs_ctx *ctx, int64_t first_pair, int64_t n_pairs);

typedef struct {
    int32_t capacity;          /* C: in-place event capacity of a 32-slot
                                  region, 32*C binary32 times.  A gate-warp
                                  whose inputs carry more than 32*C events
                                  stores its outputs in the round's spill
                                  heap instead (address in the region).  >= 1 */
    double quantum_ps;         /* 0: F mode; q > 0: Q mode, d' <- q rint(d'/q)
                                  (reading C12)                             */
    int32_t n_probe;           /* internal signals kept for readback        */
    const int32_t *probe_sig;  /* [n_probe], copied                          */
    int32_t keep_all;          /* 1: every gate output is kept (parity runs) */
    int32_t max_rerun_rounds;  /* overflow reruns; default 3.  Overflow = spill
                                  heap exhausted (rerun with a heap twice the
                                  requested size) or, with spill disabled,
                                  more than 32*C events (rerun at 4C)       */
    int32_t warps_per_cta;     /* 0: default (8)                              */
    int32_t profile;           /* 1: time the sweep kernel with CUDA events  */
    int64_t spill_bytes;       /* pass-0 spill heap: 0 = auto (the larger of
                                  arena/4, 256 MiB and 1.25x what the
                                  previous simulate on this context asked
                                  for, within free memory); > 0 = this many
                                  bytes; < 0 = no spill heap               */
    int64_t max_batch_slots;   /* slot batching (arena reused per batch):
                                  0 = auto (batch only if all slot groups'
                                  arena does not fit in device memory);
                                  > 0 = at most this many slots (rounded
                                  down to 32-slot groups) per batch.  With
                                  more than one batch, activity, latest
                                  arrival and energy cover every slot;
                                  waveforms / final values only the last
                                  batch's slots, and capture is refused.   */
    int32_t delay_in_sweep;    /* 0: a delay kernel tabulates d'(Vdd, gate,
                                  arc) in binary32 before the sweep (G x V x
                                  32 B); 1: the sweep evaluates Eq. (4)/(9)
                                  in FP64 on the fly for the gates that have
                                  observable input events ("threads
                                  of the simulation kernels independently
                                  compute modified delays on-the-fly"), no
                                  table.  Identical results.               */
} avfs_options;
avfs_status avfs_set_options(avfs_ctx *ctx, const avfs_options *opt);
avfs_status avfs_default_options(avfs_options *opt);

/* Simulate every slot in range on `cuda_stream` (cudaStream_t; NULL = the
 * legacy default stream) -- asynchronous (P:L141 step 3):
 * enqueues the delay evaluation, the stimulus expansion, the persistent
 * level-sweep kernel and the overflow check, and returns.  avfs_sync waits
 * for the work; if some slot group overflowed its waveform storage it then
 * reruns just those groups (H7) before returning, and errors (non-positive
 * delay, capacity still exceeded) are reported by avfs_sync.  Every get_*
 * call, and the next simulate, settle an outstanding simulate the same way.
 * Runs that need several slot batches settle each batch but the last
 * inside avfs_simulate.  Activity and latest arrival are accumulated over
 * the slot range and reset at the start of each call.  Returns
 * AVFS_ERR_STATE before netlist / stimuli / operating points are set, and
 * AVFS_ERR_ARG when signals x operating points (or 4 x gates x points)
 * reach 2^32 (the sweep forms its activity and delay-table rows as 32-bit
 * element offsets).                                                       */
avfs_status avfs_simulate(avfs_ctx *ctx, void *cuda_stream);
avfs_status avfs_sync(avfs_ctx *ctx);

/* ---------------------------------------------------------------- (4) */
/* Switching activity (reading C15): out[signal][n_vdd] = number of
 * transitions of the filtered waveform, summed over the simulated pairs.
 * out_is_device = 1: `out` is a device pointer (e.g. for an NCCL reduce). */
avfs_status avfs_get_activity(avfs_ctx *ctx, uint64_t *out, int32_t out_is_device);
/* Latest transition time at any primary output per operating point, max
 * over simulated pairs (Table II measurement); 0 if none.
 * out[n_vdd]; out_is_device = 1: `out` is a device pointer (a MAX reduce
 * over ranks then needs no host round trip).                              */
avfs_status avfs_get_latest_arrival(avfs_ctx *ctx, float *out, int32_t out_is_device);
/* Final logic value (init xor count parity) of signals sig[n_sig] at public
 * slots [slot0, slot0 + n_slots): out[n_sig][n_slots].  Signals must be
 * PIs, POs, probes (or any, with keep_all).                               */
avfs_status avfs_get_final_values(avfs_ctx *ctx, int32_t n_sig, const int32_t *sig,
                                  int64_t slot0, int64_t n_slots, uint8_t *out);
/* Waveforms: init[n_sig][n_slots], count[n_sig][n_slots] (true count even if
 * > cap), times[n_sig][n_slots][cap] (first min(count, cap) times, strictly
 * increasing, remaining entries 0).                                       */
avfs_status avfs_get_waveforms(avfs_ctx *ctx, int32_t n_sig, const int32_t *sig,
                               int64_t slot0, int64_t n_slots, int32_t cap,
                               uint8_t *init, int32_t *count, float *times);

/* NEXT-1 -- capture / test-response analysis (P:L141 step 4 "test
 * responses"; the frequency half of AVFS).  Every primary output
 * of every simulated pair j is sampled at the capture time t_clk[k] of its
 * operating point k: value(t) = init xor (#{t_i <= t} mod 2) (reading C1).
 * Pair j fails at k if some PO's captured value differs from its settled
 * (final) value.  Its slack is t_clk[k] - (last PO transition time), or
 * t_clk[k] if no PO switches.
 *   t_clk[n_vdd]               capture time per operating point, ps
 *   fail_pairs[n_vdd]          failing simulated pairs per point
 *   fail_po[n_po][n_vdd]       failing pairs per PO (PO order of the netlist); may be NULL
 *   slack_hist[n_vdd][n_bins]  slack histogram, bin b = [lo + b w, lo + (b+1) w),
 *                              values outside clamp to the first / last bin; may be NULL
 *   fail_bits[n_slots_sim]     1 byte per simulated public slot (stats.slots of them, in
 *                              public slot order: slot - first_slot for a slot range,
 *                              (k - 0) * n_pairs_range + (j - first_pair) for a pair
 *                              range), 1 = fails; may be NULL
 * Runs on the device over the kept PO waveforms of the last simulate.       */
avfs_status avfs_capture(avfs_ctx *ctx, const float *t_clk, int32_t n_bins, float lo_ps,
                         float width_ps, uint32_t *fail_pairs, uint32_t *fail_po,
                         uint32_t *slack_hist, uint8_t *fail_bits);

/* NEXT-4 -- switching energy per operating point (P:L37 power estimation):
 * out[k] = 1/2 sum_g act[g][k] * c_load(g) * v(g,k)^2, in fJ (c_load in fF from
 * the netlist, v(g,k) the gate's island voltage at point k, in V), summed over
 * the simulated pairs.  Gate outputs only
 * (primary inputs are driven externally).  Computed on the device.        */
avfs_status avfs_get_switching_energy(avfs_ctx *ctx, double *out_fJ);

/* NEXT-3 -- offline regression pre-process (Fig. 1 step C):
 * fit the coefficients of Eq. (4) to n characterisation samples by ordinary
 * least squares on the normal equation (Eq. 7/8), in FP64, host side.
 *   v[n], c[n]   operating points (c may be NULL iff deg_c == 0)
 *   y[n]         relative delay deviation d/d_nom - 1 (phi_D)
 *   beta[(deg_v+1)(deg_c+1)]  output, row-major [i][j] (reading C9), the
 *                layout avfs_load_library expects per (cell, pin, pol)
 *   rms          output (may be NULL): root-mean-square residual in y
 * AVFS_ERR_ARG: bad sizes / bounds, fewer samples than coefficients, or a
 * rank-deficient design matrix.                                          */
avfs_status avfs_fit_delay_polynomial(int64_t n, const double *v, const double *c, const double *y,
                                      int32_t deg_v, int32_t deg_c, double v_min, double v_max,
                                      double c_min_fF, double c_max_fF, double *beta, double *rms);

typedef struct {
    int64_t evals;               /* gates x simulated slots                  */
    int64_t slots, slot_warps;   /* simulated slots / 32-slot groups         */
    int64_t overflow_slot_warps; /* groups rerun (all rounds)                 */
    int64_t rerun_rounds;
    int64_t launches;            /* kernels launched by the last simulate    */
    int64_t arena_bytes;         /* device bytes of waveform arenas          */
    int64_t alg_bytes;           /* algorithmic bytes of the sweep */
    int32_t grid, warps_per_cta, n_scratch_buffers, n_pinned;
    double sim_ms;               /* host wall time of the last simulate      */
    double sweep_ms;             /* CUDA-event time of pass-0 sweep (profile=1) */
    int64_t spill_bytes;         /* spill-heap bytes used by the kept rounds  */
    int64_t spill_heap_bytes;    /* spill-heap bytes allocated (all rounds)   */
    int64_t batches;             /* slot batches of the last simulate         */
    int64_t enc_bytes;           /* algorithmic bytes of the stored encoding
                                    (records, entries, times)  */
    double rerun_ms;             /* CUDA-event time of the overflow reruns
                                    (profile=1), all batches                  */
} avfs_stats;
avfs_status avfs_get_stats(avfs_ctx *ctx, avfs_stats *st);

/* The CUDA-event times of the last simulate (profile=1): pass-0 sweep and
 * overflow reruns, ms.  Cheap (no readback), unlike avfs_get_stats, which
 * also derives the algorithmic bytes from the activity counters.         */
avfs_status avfs_get_timing(avfs_ctx *ctx, double *sweep_ms, double *rerun_ms);

/* Diagnostics: per-phase warp clock sums of the sweep kernel (16 counters:
 * 1 bit-parallel phase, 5 item phase, 6 level barriers), accumulated over
 * all launches since the last reset.  Only builds compiled with
 * -DAVFS_PROF_PHASES count; returns the number of counters written (0 in
 * normal builds, -1 on error).                                          */
int32_t avfs_debug_phase_cycles(uint64_t *out16, int32_t reset);

#ifdef __cplusplus
}
#endif
#endif /* AVFS_H */
