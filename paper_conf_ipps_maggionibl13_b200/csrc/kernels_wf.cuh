// Wavefront s-step kernel over the tile records (B = 1, one GPU; DESIGN.md
// sec. 5e): one launch applies s consecutive Jacobi steps (eq. 8 with
// relaxation omega, R1) to the whole vector, so the matrix records stream from
// HBM once per s steps and are re-read from L2.
//
// Work items are (step j, tile t), j = 0..s-1, listed in wave order: wave w
// holds (0, w), (1, w - L), ..., (s-1, w - (s-1) L) -- step j trails step j-1
// by a lag of L tiles -- and item i runs on CTA i mod G, each CTA in
// increasing i.  Step j of tile t reads X_j and writes X_{j+1}, the buffers
// alternating between the pass input (a.x) and the other iterate buffer
// (a.y), exactly as s single-step launches would (so the result lands where
// the double-buffer convention expects it).  Two hazards, both covered by one
// per-tile completion counter cnt[t] (each of the NCW consumer warps adds 1
// after its slice of a step j < s-1, with release semantics):
//   RAW: step j of t gathers X_j rows written by step j-1 of the tiles
//        holding them;
//   WAR: step j of t overwrites the buffer that held X_{j-1}, which step j-1
//        of the tiles reading t's rows may still gather.
// dep[t] = [first, last] tile of the union of both sets (host-computed from
// the exact rows and columns of every tile), so item (j >= 1, t) proceeds once
// cnt[u] >= NCW ((s-1) ep + j) for u in dep[t] (ep = passes before this one).
// The producer warp polls that (ld.acquire.gpu, bounded by a %globaltimer
// deadline) after issuing the tile's record copy and before the arrival that
// releases the stage to the consumers, so the acquire orders the consumers'
// gathers (mbarrier arrive/wait: release/acquire at CTA scope).  Those
// gathers are ordinary coherent loads (ld.global), never the read-only path:
// X_j is written during this grid.  L > max |dep - t| makes every dependency
// an item of an earlier wave, and all G CTAs are co-resident (G = SMs x
// occupancy), so the lowest unfinished item can always run: no deadlock.
//
// Per-row arithmetic is sell_vi2_kernel's, so every step is bit-identical to
// the single-step kernel; only the check partials' summation order differs
// (CTA c sums the rows of its last-step items).
#pragma once
#include "kernels_vi2.cuh"

namespace cme {

struct WfArgs {
    Vi2Args v;                // v.a.x = X_0 (pass input), v.a.y = the other iterate buffer
    const uint32_t* items;    // [s * n_tiles] (j << 24) | t, wave order
    const int2* dep;          // [n_tiles] {first, last} tile of RAW(t) u WAR(t)
    uint32_t* cnt;            // [n_tiles] slice-step completions (zeroed per solve)
    uint32_t* sync;           // [0] passes completed, [1] CTAs finished in this pass (zeroed per solve)
    Ctrl* ctrl;               // status CME_ERR_TIMEOUT on an expired wait
    int32_t s;                // steps per pass (2..8)
    int32_t keep;             // 1: records of steps j < s-1 stay evict_normal in L2 (else evict_first)
    int64_t timeout_ns;
};

__device__ __forceinline__ uint32_t ld_acq_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void red_release_add(uint32_t* p, uint32_t v) {
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint64_t wf_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// coherent (non read-only) gather: X_j may have been written by this grid
__device__ __forceinline__ double ld_co(const double* p) {
    double v;
    asm("ld.global.f64 %0, [%1];" : "=d"(v) : "l"(p));
    return v;
}

template <int W>
__device__ __forceinline__ double wf_row(uint32_t pv, uint32_t pc, uint32_t sdict, const double* xr) {
    double xv[W];
#pragma unroll
    for (int u = 0; u < W; ++u) xv[u] = ld_co(xr + lds_s16(pc + 64 * u));
    double acc = 0.0;
#pragma unroll
    for (int u = 0; u < W; ++u) acc = fma(lds_f64(sdict + 8 * lds_u16(pv + 64 * u)), xv[u], acc);
    return acc;
}
__device__ __forceinline__ double wf_row_wide(uint32_t pv, uint32_t pc, uint32_t sdict, const double* xr, int w) {
    double acc = 0.0;
    for (int t0 = 0; t0 < w; t0 += 8) {
        double xv[8];
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (t0 + u < w) xv[u] = ld_co(xr + lds_s16(pc + 64 * (t0 + u)));
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (t0 + u < w) acc = fma(lds_f64(sdict + 8 * lds_u16(pv + 64 * (t0 + u))), xv[u], acc);
    }
    return acc;
}

template <int NCW, bool BAND, bool REARR, bool CHECK>
__global__ void __launch_bounds__(Vi2Shape<NCW>::kThreads, Vi2Shape<NCW>::kMinBlocks)
    sell_wf_kernel(const WfArgs Wf) {
    using R = Vi2Rec<NCW, BAND, REARR>;
    const Vi2Args& V = Wf.v;
    const StepArgs& a = V.a;
    pdl_trigger();
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ uint64_t full[8], empty[8], dbar;
    __shared__ uint32_t desc[8];
    __shared__ int32_t s_stop;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int S = V.stages;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], NCW);
        }
        mbar_init(&dbar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const int G = gridDim.x, c = blockIdx.x;
    const int steps = Wf.s;
    const int n_items = steps * (int)V.n_tiles;
    const int my = c < n_items ? (n_items - 1 - c) / G + 1 : 0;
    const int pro = my < S ? my : S;
    unsigned char* stages = smem + V.dict_bytes;
    if (warp == NCW) {
        // ---------------- producer warp ----------------
        const uint64_t pol_first = evict_first_policy();
        uint64_t pol_keep;
        asm("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol_keep));
        if (lane == 0) {
            uint64_t keep;
            asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(keep));
            mbar_expect_tx(&dbar, (uint32_t)V.dict_bytes);
            bulk_g2s(smem, V.dict, (uint32_t)V.dict_bytes, &dbar, keep);
        }
        // lane l holds item k0 + l's descriptor, record offsets and dependency range
        uint32_t dsc = 0;
        int64_t o0 = 0, o1 = 0;
        int2 dp = make_int2(0, -1);
        auto load_chunk = [&](int k0) {
            const int k = k0 + lane;
            if (k < my) {
                dsc = __ldg(Wf.items + c + (int64_t)k * G);
                const int t = (int)(dsc & 0xffffffu);
                o0 = __ldg(V.rec_off + t);
                o1 = __ldg(V.rec_off + t + 1);
                dp = __ldg(Wf.dep + t);
            }
        };
        // copy of item k's record into stage s (matrix data only: no dependency)
        auto issue = [&](int k, int s) {
            const int l = k & 31;
            const int64_t b0 = __shfl_sync(0xffffffffu, o0, l), b1 = __shfl_sync(0xffffffffu, o1, l);
            const uint32_t d = __shfl_sync(0xffffffffu, dsc, l);
            if (lane == 0) {
                const int t = (int)(d & 0xffffffu), j = (int)(d >> 24);
                if (V.xpf && j == 0) {
                    const int64_t r0 = (int64_t)t * NCW * 32, r1 = min(r0 + NCW * 32, a.n_rows);
                    if (r1 > r0) prefetch_l2(a.x + a.own_off + r0, (uint64_t)(r1 - r0) * 8);
                }
                asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&full[s])),
                             "r"((uint32_t)(b1 - b0))
                             : "memory");
                bulk_g2s(stages + (size_t)s * V.stage_bytes, V.rec + b0, (uint32_t)(b1 - b0), &full[s],
                         (Wf.keep && j < steps - 1) ? pol_keep : pol_first);
            }
        };
        load_chunk(0);
        for (int k = 0; k < pro; ++k) issue(k, k);
        pdl_wait();   // X_0, cnt and sync are the previous grid's
        const bool stop = a.stop != nullptr && *(volatile const int32_t*)a.stop;
        if (lane == 0) s_stop = stop ? 1 : 0;
        if (!stop) {
            const uint32_t ep = *(volatile const uint32_t*)Wf.sync;
            bool bad = false;
            int s = 0;
            uint32_t phase = 0;
            for (int k = 0; k < my; ++k) {
                const int l = k & 31;
                if (k >= S) {   // reuse of stage s: wait for its release, then copy
                    if (l == 0) load_chunk(k);
                    mbar_wait(&empty[s], phase ^ 1u);
                    issue(k, s);
                } else if (k > 0 && l == 0) {
                    load_chunk(k);
                }
                const uint32_t d = __shfl_sync(0xffffffffu, dsc, l);
                const int j = (int)(d >> 24);
                if (j > 0 && !bad) {   // dependencies of step j: step j-1 done on dep[t]
                    const int lo = __shfl_sync(0xffffffffu, dp.x, l), hi = __shfl_sync(0xffffffffu, dp.y, l);
                    const uint32_t target = (uint32_t)NCW * ((uint32_t)(steps - 1) * ep + (uint32_t)j);
                    for (int u0 = lo; u0 <= hi; u0 += 32) {
                        const int u = u0 + lane;
                        if (u <= hi && (int32_t)(ld_acq_u32(Wf.cnt + u) - target) < 0) {
                            const uint64_t t0 = wf_ns();
                            while ((int32_t)(ld_acq_u32(Wf.cnt + u) - target) < 0) {
                                if (wf_ns() - t0 > (uint64_t)Wf.timeout_ns) { bad = true; break; }
                                __nanosleep(32);
                            }
                        }
                    }
                    bad = __any_sync(0xffffffffu, bad);
                }
                __syncwarp();
                if (lane == 0) {
                    desc[s] = d;
                    mbar_arrive(&full[s]);
                }
                if (++s == S) { s = 0; phase ^= 1u; }
            }
            if (bad && lane == 0) {
                Wf.ctrl->status = CME_ERR_TIMEOUT;
                Wf.ctrl->stop = 1;
            }
        }
        if (stop && lane == 0)   // drain the prologue copies before exit (no consumer will)
            for (int k = 0; k < pro; ++k) {
                mbar_arrive(&full[k]);
                mbar_wait(&full[k], 0u);
            }
        if (lane == 0) mbar_wait(&dbar, 0u);
        if (CHECK) cta_check_partials<NCW + 1, 1>(CheckAcc<1>(), a.partials);
        else { __syncwarp(); __syncthreads(); }
    } else {
        // ---------------- consumer warps: one slice each per item ----------------
        pdl_wait();
        CheckAcc<1> ck;
        if (!(a.stop != nullptr && *(volatile const int32_t*)a.stop)) {
            const bool damp = a.omega != 1.0;
            const double sc = a.pre_scale != nullptr ? a.pre_scale[0] : 1.0;
            const uint32_t sdict = smem_u32(smem);
            const uint32_t st0 = smem_u32(stages);
            const int n_rows = (int)a.n_rows, slice_end = (int)a.slice_end;
            const uint32_t full0 = smem_u32(full), empty0 = smem_u32(empty);
            const uint32_t sbytes = (uint32_t)V.stage_bytes;
            const uint32_t desc0 = smem_u32(desc);
            mbar_wait(&dbar, 0u);
            int s = 0;
            uint32_t phase = 0;
            uint32_t st = st0;
            for (int k = 0; k < my; ++k) {
                mbar_wait_a(full0 + 8 * s, phase);
                const uint32_t d = lds_u32(desc0 + 4 * s);
                const int t = (int)(d & 0xffffffu), j = (int)(d >> 24);
                const int q = t * NCW + warp;
                const int slot = q * 32 + lane;
                const double* xo = ((j & 1) ? a.y : a.x) + a.own_off;
                double* yo = ((j & 1) ? const_cast<double*>(a.x) : a.y) + a.own_off;
                if (q < slice_end && slot < n_rows) {
                    const int2 meta = lds_v2(st + 8 * warp);
                    const int ls = warp * 32 + lane;
                    const int r = REARR ? ((slot >> V.win_shift) << V.win_shift) + (int)lds_u8(st + R::kRow + ls) : slot;
                    const double* xr = xo + r;
                    const double x_r = ld_co(xr);
                    const uint32_t pv = st + R::kEnt + 4 * meta.x + 2 * lane;
                    const uint32_t pc = pv + 64 * meta.y;
                    double acc = 0.0;
                    switch (meta.y) {
                        case 0: break;
                        case 1: acc = wf_row<1>(pv, pc, sdict, xr); break;
                        case 2: acc = wf_row<2>(pv, pc, sdict, xr); break;
                        case 3: acc = wf_row<3>(pv, pc, sdict, xr); break;
                        case 4: acc = wf_row<4>(pv, pc, sdict, xr); break;
                        case 5: acc = wf_row<5>(pv, pc, sdict, xr); break;
                        case 6: acc = wf_row<6>(pv, pc, sdict, xr); break;
                        case 7: acc = wf_row<7>(pv, pc, sdict, xr); break;
                        case 8: acc = wf_row<8>(pv, pc, sdict, xr); break;
                        default: acc = wf_row_wide(pv, pc, sdict, xr, meta.y);
                    }
                    double sum = acc;
                    if (BAND) {
                        const double xl = ld_co(xr - 1), xu = ld_co(xr + 1);
                        const double lo = lds_f64(sdict + 8 * lds_u16(st + R::kLoUp + 2 * ls));
                        const double up = lds_f64(sdict + 8 * lds_u16(st + R::kLoUp + NCW * 64 + 2 * ls));
                        sum = fma(lo, xl, up * xu) + acc;
                    }
                    const double id = lds_f64(st + R::kInv + 8 * ls);
                    double y = damp ? fma(1.0 - a.omega, x_r, a.omega * (id * sum)) : id * sum;
                    if (j == 0) y *= sc;   // pending 1/sum(y) of the previous check (exact when sc = 1)
                    yo[r] = y;
                    if (CHECK && j == steps - 1) ck.add(0, y, x_r, id);
                }
                __syncwarp();
                if (lane == 0) {
                    if (j < steps - 1) red_release_add(Wf.cnt + t, 1u);
                    mbar_arrive_a(empty0 + 8 * s);
                }
                st += sbytes;
                if (++s == S) { s = 0; phase ^= 1u; st = st0; }
            }
        }
        if (CHECK) cta_check_partials<NCW + 1, 1>(ck, a.partials);
        else { __syncwarp(); __syncthreads(); }
    }
    // pass bookkeeping: the last CTA out counts the pass (the next pass reads
    // it after its griddepcontrol.wait, i.e. after this grid completed)
    if (threadIdx.x == 0 && !s_stop) {
        __threadfence();
        if (atomicAdd(Wf.sync + 1, 1u) == (uint32_t)G - 1) {
            Wf.sync[1] = 0;
            atomicAdd(Wf.sync, 1u);
        }
    }
}

}  // namespace cme
