/*
 * oracle/oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct FP64 event-driven logic time simulator
 * with inertial pulse cancellation, written from the paper (Schneider &
 * Wunderlich, DATE'20, /root/reference/PAPER.md, cited "P:L<n>") and the
 * readings DESIGN.md lists (C1-C17).  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load this file.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_date_schneiderw20_b200/), and never imports it.
 *
 * Operating points may give one voltage per island (NEXT-2, per-gate
 * parameters P:L155): vdd is then [point][n_isl] and gate g uses
 * vdd[k][island[g]]; n_isl = 1 is the paper's single supply.
 *
 * Functions (each cites the passage it follows):
 *   oracle_delay     -- Eq. (4), normalisations P:L117, Eq. (9) P:L135,
 *                       Horner/FMA P:L139.  Pinned by tests T1/T2/T3.
 *   oracle_sta       -- longest/shortest path arrivals (exact DAG DP) used
 *                       as the invariant of Table II.  Pinned
 *                       by brute-force path enumeration (test_oracle_sta).
 *   oracle_simulate  -- slot-parallel event-driven simulation (P:L141 steps
 *                       1-4, pin-to-pin polarity delays and inertial delay =
 *                       propagation delay P:L148; readings C1-C6, C12, C13).
 *                       Pinned by T2-T10 (closed forms, brute force, a second
 *                       independent formulation in tests/).
 *
 * No function here is "parity unpinned": O6 (flags, taint) is pinned by
 * tests/test_oracle_o6.py (windows at 0.5x / 1.5x the C13 bound for both
 * decision kinds, the truth-table exemption, soundness against a binary32
 * emulation of the method).
 *
 * Build: gcc -O2 -fopenmp -ffp-contract=off -shared -fPIC (see oracle/__init__.py).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* ------------------------------------------------------------------ */
/* O2: delay of one pin-to-pin arc at one operating point.             */
/* beta: [deg_v+1][deg_c+1] coefficients of Eq. (4) for (cell,pin,pol) */
/* x = phi_V(v) = (v - V_min)/(V_max - V_min)      */
/* z = phi_C(c) = (log2 c - log2 C_min)/(log2 C_max - log2 C_min)      */
/* f = sum_i sum_j beta_ij x^i z^j   by nested Horner with fma*/
/* d' = d_nom * (1 + f)                                   (Eq. 9)      */
/* Q mode (reading C12): d' <- q * rint(d'/q).                          */
/* ------------------------------------------------------------------ */
double oracle_delay(const double *beta, int deg_v, int deg_c, double d_nom,
                    double v, double c, double v_min, double v_max,
                    double c_min, double c_max, double quantum)
{
    double x = (v - v_min) / (v_max - v_min);
    double z = 0.0;
    if (deg_c > 0)
        z = (log2(c) - log2(c_min)) / (log2(c_max) - log2(c_min));
    double f = 0.0;
    for (int i = deg_v; i >= 0; --i) {
        /* inner Horner in z for the coefficient of x^i */
        double a = beta[i * (deg_c + 1) + deg_c];
        for (int j = deg_c - 1; j >= 0; --j)
            a = fma(a, z, beta[i * (deg_c + 1) + j]);
        f = (i == deg_v) ? a : fma(f, x, a);
    }
    double d = d_nom * (1.0 + f);
    if (quantum > 0.0)
        d = quantum * rint(d / quantum);
    return d;
}

/* ------------------------------------------------------------------ */
/* Netlist helpers (own topological sort; no levelizer shared).        */
/* ------------------------------------------------------------------ */
typedef struct {
    int32_t n_pi, n_gates, n_sig;
    const int32_t *gate_cell;
    const int64_t *fanin_ptr;
    const int32_t *fanin_sig;
    const double *d_nom;     /* [edge][2] */
    const double *c_load;    /* [gate] or NULL */
    const int32_t *cell_nin;
    const uint16_t *cell_tt;
    int32_t deg_v, deg_c;
    const double *beta;      /* [cell][4][2][deg_v+1][deg_c+1] */
    double v_min, v_max, c_min, c_max;
    const int32_t *island;   /* [gate] voltage island (NEXT-2) or NULL: island 0 */
    int32_t n_isl;           /* islands per operating point (vdd is [point][n_isl]) */
    /* derived */
    int32_t *topo;           /* gates in topological order */
    int64_t *fo_ptr;         /* fanout CSR per signal */
    int32_t *fo_gate, *fo_pin;
} Net;

static int net_prepare(Net *n)
{
    int32_t G = n->n_gates, S = n->n_sig;
    for (int32_t g = 0; g < G; ++g) {
        int64_t k = n->fanin_ptr[g + 1] - n->fanin_ptr[g];
        if (k != n->cell_nin[n->gate_cell[g]] || k < 1 || k > 4) return -2;
        for (int64_t e = n->fanin_ptr[g]; e < n->fanin_ptr[g + 1]; ++e)
            if (n->fanin_sig[e] < 0 || n->fanin_sig[e] >= S) return -2;
    }
    n->fo_ptr = calloc((size_t)S + 1, sizeof(int64_t));
    int64_t E = n->fanin_ptr[G];
    n->fo_gate = malloc(sizeof(int32_t) * (size_t)(E ? E : 1));
    n->fo_pin = malloc(sizeof(int32_t) * (size_t)(E ? E : 1));
    for (int64_t e = 0; e < E; ++e) n->fo_ptr[n->fanin_sig[e] + 1]++;
    for (int32_t s = 0; s < S; ++s) n->fo_ptr[s + 1] += n->fo_ptr[s];
    int64_t *fill = malloc(sizeof(int64_t) * (size_t)S);
    memcpy(fill, n->fo_ptr, sizeof(int64_t) * (size_t)S);
    for (int32_t g = 0; g < G; ++g)
        for (int64_t e = n->fanin_ptr[g]; e < n->fanin_ptr[g + 1]; ++e) {
            int32_t s = n->fanin_sig[e];
            n->fo_gate[fill[s]] = g;
            n->fo_pin[fill[s]] = (int32_t)(e - n->fanin_ptr[g]);
            fill[s]++;
        }
    free(fill);
    /* Kahn's algorithm on gates */
    size_t gsz = G > 0 ? (size_t)G : 1;
    int32_t *indeg = malloc(sizeof(int32_t) * gsz);
    n->topo = malloc(sizeof(int32_t) * gsz);
    int32_t head = 0, tail = 0;
    for (int32_t g = 0; g < G; ++g) {
        indeg[g] = 0;
        for (int64_t e = n->fanin_ptr[g]; e < n->fanin_ptr[g + 1]; ++e)
            if (n->fanin_sig[e] >= n->n_pi) indeg[g]++;
        if (indeg[g] == 0) n->topo[tail++] = g;
    }
    while (head < tail) {
        int32_t g = n->topo[head++];
        int32_t s = n->n_pi + g;
        for (int64_t f = n->fo_ptr[s]; f < n->fo_ptr[s + 1]; ++f)
            if (--indeg[n->fo_gate[f]] == 0) n->topo[tail++] = n->fo_gate[f];
    }
    free(indeg);
    if (tail != G) return -1;   /* cycle (O1) */
    return 0;
}

static void net_free(Net *n)
{
    free(n->topo); free(n->fo_ptr); free(n->fo_gate); free(n->fo_pin);
}

/* vrow = the operating point's island voltages; the gate uses its island's (NEXT-2) */
static double arc_delay(const Net *n, int32_t g, int32_t pin, int pol, const double *vrow, double quantum)
{
    const double v = vrow[n->island ? n->island[g] : 0];
    int32_t cell = n->gate_cell[g];
    size_t nb = (size_t)(n->deg_v + 1) * (size_t)(n->deg_c + 1);
    const double *b = n->beta + (((size_t)cell * 4 + (size_t)pin) * 2 + (size_t)pol) * nb;
    double c = n->c_load ? n->c_load[g] : 1.0;
    double dn = n->d_nom[(n->fanin_ptr[g] + pin) * 2 + pol];
    return oracle_delay(b, n->deg_v, n->deg_c, dn, v, c, n->v_min, n->v_max,
                        n->c_min, n->c_max, quantum);
}

static inline int get_bit(const uint32_t *w, int32_t i) { return (int)((w[i >> 5] >> (i & 31)) & 1u); }

/* ------------------------------------------------------------------ */
/* Longest / shortest arrival (STA-style DP, max/min over pins & pols). */
/* arr_max/arr_min: [n_vdd][n_sig]                                      */
/* ------------------------------------------------------------------ */
int oracle_sta(int32_t n_pi, int32_t n_gates, const int32_t *gate_cell,
               const int64_t *fanin_ptr, const int32_t *fanin_sig,
               const double *d_nom, const double *c_load,
               const int32_t *cell_nin, const uint16_t *cell_tt,
               int32_t deg_v, int32_t deg_c, const double *beta,
               double v_min, double v_max, double c_min, double c_max,
               int32_t n_vdd, const double *vdd, double quantum,
               const int32_t *gate_island, int32_t n_isl,
               double *arr_max, double *arr_min)
{
    Net n = {n_pi, n_gates, n_pi + n_gates, gate_cell, fanin_ptr, fanin_sig, d_nom, c_load,
             cell_nin, cell_tt, deg_v, deg_c, beta, v_min, v_max, c_min, c_max,
             gate_island, n_isl > 0 ? n_isl : 1, 0, 0, 0, 0};
    int rc = net_prepare(&n);
    if (rc) { net_free(&n); return rc; }
    for (int32_t k = 0; k < n_vdd; ++k) {
        double *amax = arr_max + (size_t)k * n.n_sig, *amin = arr_min + (size_t)k * n.n_sig;
        for (int32_t i = 0; i < n_pi; ++i) amax[i] = amin[i] = 0.0;
        for (int32_t t = 0; t < n_gates; ++t) {
            int32_t g = n.topo[t];
            double mx = -INFINITY, mn = INFINITY;
            for (int64_t e = fanin_ptr[g]; e < fanin_ptr[g + 1]; ++e) {
                int32_t pin = (int32_t)(e - fanin_ptr[g]);
                for (int pol = 0; pol < 2; ++pol) {
                    double d = arc_delay(&n, g, pin, pol, vdd + (size_t)k * n.n_isl, quantum);
                    double a = amax[fanin_sig[e]] + d, b = amin[fanin_sig[e]] + d;
                    if (a > mx) mx = a;
                    if (b < mn) mn = b;
                }
            }
            amax[n_pi + g] = mx;
            amin[n_pi + g] = mn;
        }
    }
    net_free(&n);
    return 0;
}

/* ------------------------------------------------------------------ */
/* Event queue: binary min-heap on (time, seq).                        */
/* ------------------------------------------------------------------ */
typedef struct { double t; double err; uint64_t seq; int32_t sig; int32_t val; } Ev;
typedef struct { Ev *a; int64_t n, cap; } Heap;

static int ev_less(const Ev *x, const Ev *y) { return x->t < y->t || (x->t == y->t && x->seq < y->seq); }

static void heap_push(Heap *h, Ev e)
{
    if (h->n == h->cap) { h->cap = h->cap ? 2 * h->cap : 1024; h->a = realloc(h->a, sizeof(Ev) * (size_t)h->cap); }
    int64_t i = h->n++;
    h->a[i] = e;
    while (i > 0) {
        int64_t p = (i - 1) / 2;
        if (!ev_less(&h->a[i], &h->a[p])) break;
        Ev tmp = h->a[i]; h->a[i] = h->a[p]; h->a[p] = tmp; i = p;
    }
}

static Ev heap_pop(Heap *h)
{
    Ev top = h->a[0];
    h->a[0] = h->a[--h->n];
    int64_t i = 0;
    for (;;) {
        int64_t l = 2 * i + 1, r = l + 1, m = i;
        if (l < h->n && ev_less(&h->a[l], &h->a[m])) m = l;
        if (r < h->n && ev_less(&h->a[r], &h->a[m])) m = r;
        if (m == i) break;
        Ev tmp = h->a[i]; h->a[i] = h->a[m]; h->a[m] = tmp; i = m;
    }
    return top;
}

typedef struct { int32_t gate, pin, src; double err; } Touch;

static int touch_cmp(const void *a, const void *b)
{
    const Touch *x = a, *y = b;
    if (x->gate != y->gate) return x->gate < y->gate ? -1 : 1;
    return (x->pin > y->pin) - (x->pin < y->pin);
}

/* Reading C13 (near-threshold window).  An implementation that keeps times
 * in binary32 (t32 = fl32(t32_in + fl32(d)), unit roundoff u = 2^-24) can
 * differ from the FP64 time by at most err, propagated per event:
 *   err_out = err_in (1 + u) + (1 + 2^-20) u (|d| + |t_out|)   (PI events: 0)
 * (one rounding of d to binary32, one of the sum).  Two FP64 times a, b can
 * compare differently in binary32 only if |a - b| <= err_a + err_b; such
 * decisions are flagged.  An input-order near tie is exempt when neither
 * processing order changes the gate's evaluation (all four truth-table
 * values equal), since then no output event depends on the order. */
#define U32 5.9604644775390625e-08
static inline int near(double a, double ea, double b, double eb)
{
    double w = ea + eb;
    return w > 0.0 && fabs(a - b) <= w;
}

/* ------------------------------------------------------------------ */
/* O3-O6 for a list of slots.  Slot s = (pair slot_pair[s], Vdd index  */
/* slot_vdd[s]).  Outputs for the signals out_sig[0..n_out) (NULL: all) */
/*   count [n_slots][n_out]  number of transitions (filtered waveform) */
/*   init  [n_slots][n_out]  value before t=0                          */
/*   times [n_slots][n_out][cap] first `cap` transition times (or NULL) */
/*   taint [n_slots][n_out]  near-threshold taint (F mode; or NULL)     */
/*   flags_out: number of flagged decisions (F mode)                    */
/* returns 0, -1 cycle, -2 bad arity/index, -3 non-positive delay       */
/* ------------------------------------------------------------------ */
int oracle_simulate(int32_t n_pi, int32_t n_gates, const int32_t *gate_cell,
                    const int64_t *fanin_ptr, const int32_t *fanin_sig,
                    const double *d_nom, const double *c_load,
                    const int32_t *cell_nin, const uint16_t *cell_tt,
                    int32_t deg_v, int32_t deg_c, const double *beta,
                    double v_min, double v_max, double c_min, double c_max,
                    int32_t words, const uint32_t *p1, const uint32_t *p2,
                    const double *vdd, double quantum,
                    const int32_t *gate_island, int32_t n_isl,
                    int64_t n_slots, const int64_t *slot_pair, const int32_t *slot_vdd,
                    int32_t n_out, const int32_t *out_sig, int32_t cap,
                    int32_t *count, uint8_t *init, double *times, uint8_t *taint,
                    int64_t *flags_out, int32_t n_threads)
{
    Net n = {n_pi, n_gates, n_pi + n_gates, gate_cell, fanin_ptr, fanin_sig, d_nom, c_load,
             cell_nin, cell_tt, deg_v, deg_c, beta, v_min, v_max, c_min, c_max,
             gate_island, n_isl > 0 ? n_isl : 1, 0, 0, 0, 0};
    int rc = net_prepare(&n);
    if (rc) { net_free(&n); return rc; }
    const int32_t S = n.n_sig, G = n_gates;
    if (n_out <= 0 || !out_sig) n_out = S;
    const int fmode = !(quantum > 0.0);
    int64_t flags_total = 0;
    int err = 0;
#ifdef _OPENMP
    if (n_threads > 0) omp_set_num_threads(n_threads);
#endif
#pragma omp parallel reduction(+ : flags_total)
    {
        uint8_t *val = malloc((size_t)S);
        uint8_t *init_v = malloc((size_t)S);
        uint32_t *inbits = malloc(sizeof(uint32_t) * (size_t)(G ? G : 1));
        uint8_t *proj = malloc((size_t)(G ? G : 1));
        uint64_t *pend = malloc(sizeof(uint64_t) * (size_t)(G ? G : 1));
        double *pend_t = malloc(sizeof(double) * (size_t)(G ? G : 1));
        double *pend_e = malloc(sizeof(double) * (size_t)(G ? G : 1));
        double *last_oe = malloc(sizeof(double) * (size_t)(G ? G : 1));
        double *last_ie = malloc(sizeof(double) * (size_t)(G ? G : 1));
        double *last_out = malloc(sizeof(double) * (size_t)(G ? G : 1));
        double *last_in = malloc(sizeof(double) * (size_t)(G ? G : 1));
        int32_t *last_src = malloc(sizeof(int32_t) * (size_t)(G ? G : 1));
        int32_t *last_pin = malloc(sizeof(int32_t) * (size_t)(G ? G : 1));
        uint8_t *flag = malloc((size_t)(G ? G : 1));
        uint8_t *tnt = malloc((size_t)S);
        int32_t *cnt = malloc(sizeof(int32_t) * (size_t)S);
        int32_t *wcap = malloc(sizeof(int32_t) * (size_t)S);      /* per-signal time storage */
        double **wt = calloc((size_t)S, sizeof(double *));
        Heap heap = {0, 0, 0};
        Touch *touch = NULL; int64_t touch_cap = 0;

#pragma omp for schedule(dynamic, 1)
        for (int64_t s = 0; s < n_slots; ++s) {
            const int64_t j = slot_pair[s];
            const double *v = vdd + (size_t)slot_vdd[s] * n.n_isl;   /* island voltages */
            const uint32_t *w1 = p1 + (size_t)j * (size_t)words, *w2 = p2 + (size_t)j * (size_t)words;
            /* O3: static evaluation of p1 in topological order */
            for (int32_t i = 0; i < n_pi; ++i) val[i] = (uint8_t)get_bit(w1, i);
            for (int32_t t = 0; t < G; ++t) {
                int32_t g = n.topo[t];
                uint32_t b = 0;
                for (int64_t e = fanin_ptr[g]; e < fanin_ptr[g + 1]; ++e)
                    b |= (uint32_t)val[fanin_sig[e]] << (e - fanin_ptr[g]);
                val[n_pi + g] = (uint8_t)((cell_tt[gate_cell[g]] >> b) & 1u);
            }
            memcpy(init_v, val, (size_t)S);
            for (int32_t g = 0; g < G; ++g) {
                uint32_t b = 0;
                for (int64_t e = fanin_ptr[g]; e < fanin_ptr[g + 1]; ++e)
                    b |= (uint32_t)val[fanin_sig[e]] << (e - fanin_ptr[g]);
                inbits[g] = b;
                proj[g] = val[n_pi + g];
                pend[g] = 0; pend_t[g] = 0.0; pend_e[g] = 0.0;
                last_out[g] = -INFINITY; last_oe[g] = 0.0;
                last_in[g] = -INFINITY; last_ie[g] = 0.0; last_src[g] = -1; last_pin[g] = 0;
                flag[g] = 0;
            }
            for (int32_t i = 0; i < S; ++i) { cnt[i] = 0; }
            heap.n = 0;
            uint64_t seq = 1;
            /* C2: PI i transitions at t = 0 iff p1 != p2 */
            for (int32_t i = 0; i < n_pi; ++i)
                if (get_bit(w1, i) != get_bit(w2, i))
                    heap_push(&heap, (Ev){0.0, 0.0, seq++, i, get_bit(w2, i)});
            /* O4: process distinct times in increasing order */
            while (heap.n > 0) {
                const double t = heap.a[0].t;
                int64_t nt = 0;
                /* O4.1: mature every non-cancelled event at t */
                while (heap.n > 0 && heap.a[0].t == t) {
                    Ev e = heap_pop(&heap);
                    if (e.sig >= n_pi) {
                        int32_t g = e.sig - n_pi;
                        if (pend[g] != e.seq) continue;          /* cancelled */
                        pend[g] = 0;
                        last_out[g] = t;
                        last_oe[g] = e.err;
                    }
                    val[e.sig] = (uint8_t)e.val;
                    int32_t c = cnt[e.sig]++;
                    if (c >= (wt[e.sig] ? wcap[e.sig] : 0)) {
                        int32_t nc = wt[e.sig] ? 2 * wcap[e.sig] : 4;
                        wt[e.sig] = realloc(wt[e.sig], sizeof(double) * (size_t)nc);
                        wcap[e.sig] = nc;
                    }
                    wt[e.sig][c] = t;
                    for (int64_t f = n.fo_ptr[e.sig]; f < n.fo_ptr[e.sig + 1]; ++f) {
                        if (nt == touch_cap) { touch_cap = touch_cap ? 2 * touch_cap : 256; touch = realloc(touch, sizeof(Touch) * (size_t)touch_cap); }
                        touch[nt++] = (Touch){n.fo_gate[f], n.fo_pin[f], e.sig, e.err};
                    }
                }
                /* O4.2: per touched gate, ascending pin order (reading C5) */
                qsort(touch, (size_t)nt, sizeof(Touch), touch_cmp);
                for (int64_t i = 0; i < nt; ++i) {
                    const int32_t g = touch[i].gate, p = touch[i].pin;
                    if (fmode) {     /* O6: input-order near tie on different sources */
                        if (last_src[g] >= 0 && last_src[g] != touch[i].src &&
                            near(t, touch[i].err, last_in[g], last_ie[g])) {
                            /* b = inputs after the previous event A, before this event B */
                            const uint32_t b = inbits[g], A = 1u << last_pin[g], B = 1u << p;
                            const uint16_t tt = cell_tt[gate_cell[g]];
                            const uint32_t y0 = (tt >> (b ^ A)) & 1u, yA = (tt >> b) & 1u;
                            const uint32_t yB = (tt >> (b ^ A ^ B)) & 1u, yAB = (tt >> (b ^ B)) & 1u;
                            if (!(y0 == yA && y0 == yB && y0 == yAB)) { flag[g] = 1; flags_total++; }
                        }
                        last_in[g] = t; last_ie[g] = touch[i].err; last_src[g] = touch[i].src; last_pin[g] = p;
                    }
                    inbits[g] ^= 1u << p;
                    const int y = (int)((cell_tt[gate_cell[g]] >> inbits[g]) & 1u);
                    if (y == proj[g]) continue;                 /* O4.3 / C4 */
                    if (fmode) {     /* O6: filter-decision margin */
                        double tl = pend[g] ? pend_t[g] : last_out[g];
                        double el = pend[g] ? pend_e[g] : last_oe[g];
                        if (tl > -INFINITY && near(tl, el, t, touch[i].err)) { flag[g] = 1; flags_total++; }
                    }
                    if (pend[g]) {                               /* O4.4 / C3: cancel */
                        pend[g] = 0;
                        proj[g] = (uint8_t)y;
                    } else {                                     /* O4.5: schedule */
                        double d = arc_delay(&n, g, p, y, v, quantum);
                        if (!(d > 0.0)) {
#pragma omp atomic write
                            err = -3;
                            d = 1.0;
                        }
                        double tn = t + d;
                        double en = fmode ? touch[i].err * (1.0 + U32) + (1.0 + 0x1p-20) * U32 * (fabs(d) + fabs(tn)) : 0.0;
                        pend[g] = seq;
                        pend_t[g] = tn;
                        pend_e[g] = en;
                        heap_push(&heap, (Ev){tn, en, seq++, n_pi + g, y});
                        proj[g] = (uint8_t)y;
                    }
                }
            }
            /* O6 taint propagation in topological order */
            for (int32_t i = 0; i < n_pi; ++i) tnt[i] = 0;
            for (int32_t t = 0; t < G; ++t) {
                int32_t g = n.topo[t];
                uint8_t x = flag[g];
                for (int64_t e = fanin_ptr[g]; e < fanin_ptr[g + 1]; ++e) x |= tnt[fanin_sig[e]];
                tnt[n_pi + g] = x;
            }
            /* O5: outputs */
            for (int32_t o = 0; o < n_out; ++o) {
                int32_t sg = out_sig ? out_sig[o] : o;
                size_t idx = (size_t)s * (size_t)n_out + (size_t)o;
                count[idx] = cnt[sg];
                init[idx] = init_v[sg];
                if (taint) taint[idx] = tnt[sg];
                if (times && cap > 0) {
                    double *dst = times + idx * (size_t)cap;
                    for (int32_t c = 0; c < cap; ++c) dst[c] = c < cnt[sg] ? wt[sg][c] : 0.0;
                }
            }
        }
        for (int32_t i = 0; i < S; ++i) free(wt[i]);
        free(wt); free(wcap); free(cnt); free(tnt); free(flag); free(last_src); free(last_pin); free(last_in);
        free(last_out); free(pend_t); free(pend_e); free(last_oe); free(last_ie); free(pend); free(proj); free(inbits); free(init_v); free(val);
        free(heap.a); free(touch);
    }
    net_free(&n);
    if (flags_out) *flags_out = flags_total;
    return err;
}

int oracle_max_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
