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
// Per-slot merge of up to K sorted input event lists with the inertial filter
// (reading C3: cancel the pending last output event iff it lies strictly after
// the input event; C4: no reschedule on confirming events; C5: ties in time
// are taken in ascending pin order).  Returns the exact output count; the
// first `cstage` surviving events are left in s_out[i*32 + lane].
// ---------------------------------------------------------------------------
template <int K>
__device__ __forceinline__ int merge_slot(const float* __restrict__ s_in, const int (&c0)[KMAX],
                                          const int (&n)[KMAX], const bool (&pi)[KMAX],
                                          const float (&df)[KMAX], const float (&dr)[KMAX],
                                          uint32_t tt, uint32_t bits, uint32_t proj,
                                          float* __restrict__ s_out, int cstage, int lane) {
    const float INF = __int_as_float(0x7f800000);
    float h[K];
    int c[K], e[K];
#pragma unroll
    for (int q = 0; q < K; ++q) {
        c[q] = pi[q] ? 0 : c0[q];
        e[q] = c[q] + n[q];
        h[q] = (n[q] > 0) ? (pi[q] ? 0.0f : s_in[c[q]]) : INF;
    }
    int n_out = 0;
    float tl = -INF;
    for (;;) {
        float t = h[0];
        int pm = 0;
#pragma unroll
        for (int q = 1; q < K; ++q)
            if (h[q] < t) { t = h[q]; pm = q; }
        if (!(t < INF)) break;
        int cn = c[0], en = e[0];
        float d_r = dr[0], d_f = df[0];
#pragma unroll
        for (int q = 1; q < K; ++q)
            if (q == pm) { cn = c[q]; en = e[q]; d_r = dr[q]; d_f = df[q]; }
        ++cn;
        const float hn = (cn < en) ? s_in[cn] : INF;
#pragma unroll
        for (int q = 0; q < K; ++q)
            if (q == pm) { c[q] = cn; h[q] = hn; }
        bits ^= 1u << pm;
        const uint32_t y = (tt >> bits) & 1u;
        if (y != proj) {
            proj = y;
            if (tl > t) {            // pending output lies after t: pulse filtered
                --n_out;
                tl = -INF;           // the event before it is <= t (never cancelled twice)
            } else {
                tl = t + (y ? d_r : d_f);
                if (n_out < cstage) s_out[n_out * 32 + lane] = tl;
                ++n_out;
            }
        }
    }
    return n_out;
}

__device__ __forceinline__ uint8_t* region_of(uint32_t loc, uint8_t* scr, int64_t scr_stride,
                                              uint8_t* pin, int64_t pin_stride) {
    const int64_t id = loc & LOC_ID;
    return ((loc & LOC_KIND) == LOC_SCRATCH) ? scr + id * scr_stride : pin + id * pin_stride;
}

__global__ void __launch_bounds__(512) sweep_kernel(const SweepParams p) {
    extern __shared__ __align__(16) float smem[];
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    const int nw = blockDim.x >> 5;
    const int in_words = p.kmax * p.W + 16;
    float* s_in = smem + (size_t)warp * (size_t)(in_words + 32 * p.cstage);
    float* s_out = s_in + in_words;
    const bool first_pass = (p.prev_W == 0);
    const int64_t scr_stride = (int64_t)gridDim.x * p.region_bytes;
    const int64_t pin_stride = p.n_sw * p.region_bytes;

    for (int64_t i = blockIdx.x; i < p.n_sw; i += gridDim.x) {
        const int64_t sw = p.sw_list ? (int64_t)p.sw_list[i] : p.sw_first + i;
        const int kv = (int)(sw / p.n_pw);
        const int pw = (int)(sw % p.n_pw);
        const int64_t j = (int64_t)pw * 32 + lane;
        const int64_t pub = (int64_t)kv * p.n_pairs + j;
        const bool valid = j < p.n_pairs && pub >= p.slot_first && pub < p.slot_end;
        const uint32_t mask = __ballot_sync(0xffffffffu, valid);
        // Step 2: the operating point of this slot group, normalised
        const double x = (p.vdd[kv] - p.v_min) / (p.v_max - p.v_min);
        uint8_t* scr = p.scratch + (int64_t)blockIdx.x * p.region_bytes;
        uint8_t* pin = p.pinned + i * p.region_bytes;

        for (int L = 0; L < p.depth; ++L) {
            const int g_end = p.level_ptr[L + 1];
            for (int gi = p.level_ptr[L] + warp; gi < g_end; gi += nw) {
                const GateDesc* G = p.gates + gi;
                // Step 1: gate description, warp-uniform
                const uint4 ins = __ldg(reinterpret_cast<const uint4*>(G));
                const uint4 hd = __ldg(reinterpret_cast<const uint4*>(G) + 1);
                const uint32_t out_loc = hd.x, sig = hd.y;
                const uint32_t tt = hd.z & 0xffffu;
                const int K = (int)((hd.z >> 16) & 0xffu);
                const uint32_t gflags = hd.z >> 24;
                // Steps 3-5, repeated per pin-to-pin delay: lane
                // 2*pin+pol evaluates Eq. (4) by Horner/FMA in FP64 and Eq. (9)
                float dl = 1.0f;
                if (lane < 2 * K) {
                    const double* cf = p.coef + hd.w + lane * (p.deg_v + 1);
                    double f = __ldg(cf + p.deg_v);
                    for (int t = p.deg_v - 1; t >= 0; --t) f = fma(f, x, __ldg(cf + t));
                    double d = __ldg(&G->dnom[lane]) * (1.0 + f);
                    if (p.quantum > 0.0) d = p.quantum * rint(d / p.quantum);
                    if (!(d > 0.0)) atomicOr(p.err, 1);
                    dl = __double2float_rn(d);
                }
                float df[KMAX], dr[KMAX];
#pragma unroll
                for (int q = 0; q < KMAX; ++q) {
                    df[q] = __shfl_sync(0xffffffffu, dl, 2 * q);
                    dr[q] = __shfl_sync(0xffffffffu, dl, 2 * q + 1);
                }
                // input waveforms: headers (coalesced) or PI bits (broadcast)
                const uint32_t in_loc[KMAX] = {ins.x, ins.y, ins.z, ins.w};
                int n[KMAX];
                bool isp[KMAX];
                const float* ev[KMAX];
                uint32_t bits = 0, pois = 0, prevp = 0;
#pragma unroll
                for (int q = 0; q < KMAX; ++q) {
                    n[q] = 0;
                    isp[q] = true;
                    ev[q] = nullptr;
                    if (q < K) {
                        const uint32_t loc = in_loc[q];
                        if ((loc & LOC_KIND) == LOC_PI) {
                            const int64_t o = (int64_t)(loc & LOC_ID) * p.n_pw + pw;
                            const uint32_t w1 = __ldg(p.p1t + o) & mask;
                            const uint32_t w2 = __ldg(p.p2t + o) & mask;
                            bits |= ((w1 >> lane) & 1u) << q;
                            n[q] = (int)(((w1 ^ w2) >> lane) & 1u);
                        } else {
                            const uint8_t* r = region_of(loc, scr, scr_stride, pin, pin_stride);
                            const uint32_t h = ld_u32(r + 4 * lane);
                            n[q] = (int)(h & HDR_N);
                            bits |= ((h >> 20) & 1u) << q;
                            pois |= h & HDR_POISON;
                            prevp |= h & HDR_PREV;
                            isp[q] = false;
                            ev[q] = reinterpret_cast<const float*>(r + 128);
                        }
                    }
                }
                const uint32_t y0 = (tt >> bits) & 1u;
                uint8_t* ro = region_of(out_loc, scr, scr_stride, pin, pin_stride);
                uint32_t* ro_hdr = reinterpret_cast<uint32_t*>(ro);
                const bool any_prev = __any_sync(0xffffffffu, prevp != 0);
                if (__any_sync(0xffffffffu, pois != 0)) {
                    ro_hdr[lane] = HDR_POISON | HDR_PREV | (y0 << 20);
                    continue;
                }
                // compact per-pin offsets: exclusive warp scans of the counts
                int c0[KMAX], tot[KMAX];
                {
                    const uint32_t a = (uint32_t)(isp[0] ? 0 : n[0]) | ((uint32_t)(isp[1] ? 0 : n[1]) << 16);
                    const uint32_t ia = warp_incl_scan(a, lane);
                    const uint32_t ta = __shfl_sync(0xffffffffu, ia, 31);
                    const uint32_t ea = ia - a;
                    c0[0] = (int)(ea & 0xffffu);  tot[0] = (int)(ta & 0xffffu);
                    c0[1] = (int)(ea >> 16);      tot[1] = (int)(ta >> 16);
                    if (K > 2) {
                        const uint32_t b = (uint32_t)(isp[2] ? 0 : n[2]) | ((uint32_t)(isp[3] ? 0 : n[3]) << 16);
                        const uint32_t ib = warp_incl_scan(b, lane);
                        const uint32_t tb = __shfl_sync(0xffffffffu, ib, 31);
                        const uint32_t eb = ib - b;
                        c0[2] = (int)(eb & 0xffffu);  tot[2] = (int)(tb & 0xffffu);
                        c0[3] = (int)(eb >> 16);      tot[3] = (int)(tb >> 16);
                    } else {
                        c0[2] = c0[3] = tot[2] = tot[3] = 0;
                    }
                }
                // stage the compact input lists into shared memory (16-B cp.async)
                int base = 0;
#pragma unroll
                for (int q = 0; q < KMAX; ++q) {
                    if (q < K && !isp[q]) {
                        const int nv = (tot[q] + 3) >> 2;
                        for (int v = lane; v < nv; v += 32) cp_async16(s_in + base + 4 * v, ev[q] + 4 * v);
                        c0[q] += base;
                        base += nv * 4;
                    }
                }
                cp_async_wait_all();
                __syncwarp();
                int n_out;
                switch (K) {
                    case 1: n_out = merge_slot<1>(s_in, c0, n, isp, df, dr, tt, bits, y0, s_out, p.cstage, lane); break;
                    case 2: n_out = merge_slot<2>(s_in, c0, n, isp, df, dr, tt, bits, y0, s_out, p.cstage, lane); break;
                    case 3: n_out = merge_slot<3>(s_in, c0, n, isp, df, dr, tt, bits, y0, s_out, p.cstage, lane); break;
                    default: n_out = merge_slot<4>(s_in, c0, n, isp, df, dr, tt, bits, y0, s_out, p.cstage, lane); break;
                }
                // output: scan, overflow ballot, compaction, 128-bit stores
                const uint32_t incl = warp_incl_scan((uint32_t)n_out, lane);
                const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
                const uint32_t excl = incl - (uint32_t)n_out;
                const bool ovf = __any_sync(0xffffffffu, n_out > p.cstage) || total > (uint32_t)p.W;
                bool prev = true;
                if (!first_pass)
                    prev = any_prev || __any_sync(0xffffffffu, n_out > p.prev_cstage) || total > (uint32_t)p.prev_W;
                __syncwarp();
                if (!ovf) {
                    for (int t = 0; t < n_out; ++t) s_in[excl + t] = s_out[t * 32 + lane];
                    __syncwarp();
                    float* dst = reinterpret_cast<float*>(ro + 128);
                    const int nv = (int)((total + 3) >> 2);
                    for (int v = lane; v < nv; v += 32)
                        st_global_v4(dst + 4 * v, reinterpret_cast<const float4*>(s_in)[v]);
                } else if (lane == 0) {
                    p.ovf[i] = 1;
                }
                ro_hdr[lane] = (uint32_t)min(n_out, (int)HDR_N) | (y0 << 20) | (ovf ? HDR_POISON : 0u) |
                               (prev ? HDR_PREV : 0u);
                // activity (reading C15) and latest PO arrival: counted
                // once per slot across overflow rounds (only where prev && !ovf)
                if (!ovf && prev) {
                    if (lane == 0 && total) atomicAdd(p.act + (int64_t)sig * p.n_vdd + kv, (unsigned long long)total);
                    if (gflags & 1u) {
                        const float last = n_out ? s_out[(n_out - 1) * 32 + lane] : 0.0f;
                        const uint32_t m = __reduce_max_sync(0xffffffffu, __float_as_uint(last));
                        if (lane == 0 && m) atomicMax(p.latest + kv, m);
                    }
                }
                __syncwarp();
            }
            __syncthreads();
        }
    }
}

int sweep_smem_bytes(int warps_per_cta, int kmax, int W, int cstage) {
    return warps_per_cta * (kmax * W + 16 + 32 * cstage) * 4;
}

cudaError_t sweep_occupancy(int warps_per_cta, int smem, int* blocks_per_sm) {
    cudaError_t e = cudaFuncSetAttribute(sweep_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, sweep_kernel, warps_per_cta * 32, smem);
}

cudaError_t launch_sweep(const SweepParams& p, int grid, int warps_per_cta, cudaStream_t st) {
    const int smem = sweep_smem_bytes(warps_per_cta, p.kmax, p.W, p.cstage);
    cudaError_t e = cudaFuncSetAttribute(sweep_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    sweep_kernel<<<grid, warps_per_cta * 32, smem, st>>>(p);
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
        init = (h >> 20) & 1u;
        n = (int)(h & HDR_N);
        int off = 0;
        for (int l = 0; l < lane; ++l) off += (int)(hdr[l] & HDR_N);
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

}  // namespace avfs
