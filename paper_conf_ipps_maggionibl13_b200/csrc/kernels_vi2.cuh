// Tile-record value-indexed step kernel (B = 1): the hot
// kernel on the toggle-switch CMEs.  Same operator and arithmetic as
// sell_vi_kernel -- y = (1-omega) x + omega inv_d (sum_t dict[vidx] x[r + col])
// (eq. 8, R1), FMAs in t order, row sum times inv_d -- so its results
// are bit-identical to it and to the layout-v0 kernels.  What changes is how
// the encoding reaches the SM and how lean the consumer loop is:
//
// * Tile records.  Everything a tile needs is ONE contiguous record in HBM --
//   [slice metadata | row8 | loi, upi | inv_d | per slice: vidx block, col16
//   block] -- moved by ONE cp.async.bulk per tile.  sell_vi_kernel issued 4-6
//   bulk copies per tile (metadata 128 B, row8 512 B, ...) plus a separate
//   per-lane inv_d stream, and its TMA ring alone (consumers idle: CME_ABL=1)
//   topped out at 5.4 TB/s of DRAM reads.
// * inv_d comes from shared memory (no global load on the slice's critical
//   path besides the x gathers).
// * All stage addressing is 32-bit shared-window arithmetic derived from the
//   slice's {entry offset, width} record; omega and the buffer pointers stay
//   kernel parameters (constant-bank operands), so the consumer loop fits the
//   40-register budget of 2 x 24-warp CTAs per SM (46 consumer warps) where
//   sell_vi_kernel needs 56 (32 warps).  Measured: the step is bound by the
//   latency of the x gathers behind one shared-memory round trip, so resident
//   consumer warps set the rate.
#pragma once
#include "kernels_cpt.cuh"

namespace cme {

// Fused peer-memory halo synchronisation (row-sharded solve, peer-memory
// transport): instead of a flag-barrier kernel after every
// step, the step kernel itself orders the halo traffic of the boundary tiles.
// Per step k (= local[0], steps this rank has run; every rank runs the same
// sequence) and neighbour pair:
//   RAW  a tile reading halo rows waits until every rank pushing to me has
//        signalled pushed >= k (its step k-1 stores of x_k into my buffer);
//   WAR  a tile pushing rows waits until every rank I push to has signalled
//        consumed >= k (its step k-1 reads of the buffer I now overwrite).
// The waits gate the producer's stage arrival (the consumers never see a
// gated tile early); the signals go out when the last warp of the last
// push (halo) tile of the step finishes: atomic count at gpu scope, then
// fence.sc.sys and st.release.sys of k+1 into the peers' flag words.  All
// spins are bounded (%globaltimer): CME_ERR_TIMEOUT, never a hung GPU.
struct HaloSync {
    int64_t* local;                          // [0] steps run, [1] push-warp and [2] halo-warp completions, [3] CTAs out
    const int64_t* pushed;                   // [nranks] written by the ranks pushing to me
    const int64_t* consumed;                 // [nranks] written by the ranks I push to
    int64_t* peer_pushed[kMaxPushPeers];     // send peer's pushed[my rank]
    int64_t* peer_consumed[kMaxPushPeers];   // recv peer's consumed[my rank]
    int32_t send_rank[kMaxPushPeers], recv_rank[kMaxPushPeers];
    int32_t nsend, nrecv;
    const uint8_t* tile_kind;                // [tiles] bit 0: reads halo rows, bit 1: pushes rows
    int64_t push_warps, halo_warps;          // consumer-warp slots per step in push / halo tiles
    int64_t timeout_ns;
    Ctrl* ctrl;
    int32_t on;
};

__device__ __forceinline__ int64_t ld_acquire_sys_s64(const int64_t* p) {
    int64_t v;
    asm volatile("ld.acquire.sys.global.s64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t hs_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// producer warp: wait for the peers' flags tile kind `kind` depends on (all lanes call)
static __device__ __noinline__ void hs_gate(const HaloSync& hs, uint32_t kind, int64_t k, bool& bad) {
    const int lane = threadIdx.x & 31;
    const int64_t* f = nullptr;
    if ((kind & 1u) && lane < hs.nrecv) f = hs.pushed + hs.recv_rank[lane];
    if ((kind & 2u) && lane >= 16 && lane - 16 < hs.nsend) f = hs.consumed + hs.send_rank[lane - 16];
    if (f != nullptr && !bad && ld_acquire_sys_s64(f) < k) {
        const uint64_t t0 = hs_ns();
        while (ld_acquire_sys_s64(f) < k) {
            if (hs_ns() - t0 > (uint64_t)hs.timeout_ns) { bad = true; break; }
            __nanosleep(64);
        }
    }
    bad = __any_sync(0xffffffffu, bad);
}
__device__ __forceinline__ int64_t atom_add_acq_rel(int64_t* p, int64_t v) {
    int64_t old;
    asm volatile("atom.acq_rel.gpu.global.add.u64 %0, [%1], %2;" : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
}
// consumer lane 0 after its slice of a push / halo tile of step k (after a
// __syncwarp: the lanes' peer stores / halo reads precede the release)
static __device__ __noinline__ void hs_signal(const HaloSync& hs, uint32_t kind, int64_t k) {
    if (kind & 2u) {
        const int64_t old = atom_add_acq_rel(hs.local + 1, 1);
        if ((int64_t)old + 1 == (k + 1) * hs.push_warps) {   // last push slice of the step
            __threadfence_system();
            for (int p = 0; p < hs.nsend; ++p)
                asm volatile("st.release.sys.global.s64 [%0], %1;" ::"l"(hs.peer_pushed[p]), "l"(k + 1) : "memory");
        }
    }
    if (kind & 1u) {
        const int64_t old = atom_add_acq_rel(hs.local + 2, 1);
        if ((int64_t)old + 1 == (k + 1) * hs.halo_warps) {   // last halo-reading slice of the step
            __threadfence_system();
            for (int q = 0; q < hs.nrecv; ++q)
                asm volatile("st.release.sys.global.s64 [%0], %1;" ::"l"(hs.peer_consumed[q]), "l"(k + 1) : "memory");
        }
    }
}

// end of a step kernel (all threads): the last CTA out counts the step (the
// next step reads it after its griddepcontrol.wait); stopped launches do not
__device__ __forceinline__ void hs_finish(const HaloSync& hs, int G, const int32_t* stop) {
    __syncwarp();
    __syncthreads();
    if (threadIdx.x == 0 && !(stop != nullptr && *(volatile const int32_t*)stop)) {
        __threadfence();
        if (atomicAdd(reinterpret_cast<unsigned long long*>(hs.local + 3), 1ull) == (unsigned long long)G - 1) {
            hs.local[3] = 0;
            __threadfence();
            atomicAdd(reinterpret_cast<unsigned long long*>(hs.local), 1ull);
        }
    }
}

struct Vi2Args {
    StepArgs a;              // n_rows, slice_end, x/y, own_off, omega, pre_scale, partials, stop, inv_d (checks), push
    const unsigned char* rec;   // tile records, rec_off[t] bytes from rec
    const int64_t* rec_off;     // [n_tiles + 1]
    const double* dict;         // [dict_bytes / 8], 128-B padded
    int64_t n_tiles;
    int32_t stages;
    int32_t stage_bytes;        // >= the largest record, multiple of 128
    int32_t dict_bytes;
    int32_t win_shift;          // log2(rearrangement window) (REARR)
    int32_t xpf;                // L2 prefetch of each tile's own x rows with its record
    HaloSync hs;                // fused halo synchronisation (hs.on = 0: none)
    // x window in shared memory (XW kernels): chunk k of
    // the ring holds the iterate rows [256 k - xw_off, 256 k - xw_off + 256)
    // (relative to x + own_off) at ring slot k mod NX (NX = xw_rows / 256),
    // and slots 0 .. xw_mirror-1 again at NX .. NX+xw_mirror-1, so that a
    // tile's chunks are contiguous in shared memory (no wrap in the gathers);
    // tile t needs chunks [xw_ch[t].x, xw_ch[t].y) (suffix-min / prefix-max)
    const int2* xw_ch;
    int32_t xw_rows;            // ring rows (a multiple of 256) without the mirror
    int32_t xw_mirror;          // mirrored chunks (>= the widest tile's chunks - 1)
    int32_t xw_off;             // 1: x + own_off is 8 mod 16 (bulk copies need 16-B sources; row -1 loadable)
    int64_t xw_nx;              // iterate rows readable from x + own_off (a sentinel row at -1 and nx)
    int32_t contig;             // gather kernels: contiguous tile ranges per CTA (CME_VI2_CONTIG) instead of c + i G
};

// Record layout of a tile of TS slices (byte offsets; every block 16-B aligned).
// F64 (ENC = 2, the compact encoding of sec. 5b, no value index): lo/up are
// M's band values (double), no inv_d block (only CHECK/transient steps read
// inv_d, from global memory), and a slice's entries are val_c[32 W] (double)
// then col16[32 W].
template <int TS, bool BAND, bool REARR, bool F64 = false>
struct Vi2Rec {
    static constexpr int kMeta = ((TS + 1) & ~1) * 8;              // int2 {entry offset, width} per slice
    static constexpr int kRow = kMeta;                            // uint8 per slot (REARR)
    static constexpr int kLoUp = kRow + (REARR ? TS * 32 : 0);    // uint16 loi, upi (F64: double lo, up) per slot (BAND)
    static constexpr int kInv = kLoUp + (BAND ? TS * (F64 ? 512 : 128) : 0);   // double per slot (not F64)
    static constexpr int kEnt = kInv + (F64 ? 0 : TS * 256);      // per slice: vidx (F64: val_c) [32 W] then col16[32 W]
    static constexpr int kEntBytes = F64 ? 10 : 4;                // bytes per entry
};
__host__ __device__ constexpr int vi2_fixed_bytes(int ts, bool band, bool rearr, bool f64 = false) {
    return ((ts + 1) & ~1) * 8 + (rearr ? ts * 32 : 0) + (band ? ts * (f64 ? 512 : 128) : 0) + (f64 ? 0 : ts * 256);
}

__device__ __forceinline__ uint32_t lds_u16(uint32_t a) {
    uint16_t v;
    asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ int32_t lds_s16(uint32_t a) {
    int16_t v;
    asm volatile("ld.shared.s16 %0, [%1];" : "=h"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint32_t lds_u8(uint32_t a) {
    uint16_t v;
    asm volatile("ld.shared.u8 %0, [%1];" : "=h"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ double lds_f64(uint32_t a) {
    double v;
    asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint32_t lds_u32(uint32_t a) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
// mbarrier wait / arrive on a 32-bit shared-window address (no generic ->
// shared conversion in the loop)
__device__ __forceinline__ void mbar_wait_a(uint32_t b, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, %2;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" ::"r"(b),
        "r"(parity), "n"(CME_MBAR_SUSPEND_NS)
        : "memory");
}
__device__ __forceinline__ void mbar_arrive_a(uint32_t b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(b) : "memory");
}
__device__ __forceinline__ int2 lds_v2(uint32_t a) {
    int2 v;
    asm volatile("ld.shared.v2.s32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
    return v;
}

// x gathers: from global memory (L1/L2; the iterate row r is xr[0]) or from
// the shared-memory x window (XW)
struct GatherG {
    const double* xr;
    __device__ __forceinline__ double operator()(int32_t o) const { return __ldg(xr + o); }
};
struct GatherS {
    uint32_t xr;     // shared-window address of row r in the (mirrored) ring
    __device__ __forceinline__ double operator()(int32_t o) const { return lds_f64(xr + ((uint32_t)o << 3)); }
};
struct GatherW {     // ring without the mirror: one conditional wrap per entry
    uint32_t xr;     // shared-window address of row r before the wrap
    int32_t lim;     // offsets o >= lim lie past the ring's end (X - ring index of row r)
    uint32_t back;   // 8 X
    __device__ __forceinline__ double operator()(int32_t o) const {
        const uint32_t a = xr + ((uint32_t)o << 3);
        return lds_f64(o >= lim ? a - back : a);
    }
};

// W entries of one slot: the W x gathers first (their latency is the step's
// critical path), then per entry the dictionary value and the FMA in t order.
template <int W, class GX>
__device__ __forceinline__ double vi2_row(uint32_t pv, uint32_t pc, uint32_t sdict, const GX& gx) {
    double xv[W];
#pragma unroll
    for (int u = 0; u < W; ++u) xv[u] = gx(lds_s16(pc + 64 * u));
    double acc = 0.0;
#pragma unroll
    for (int u = 0; u < W; ++u) acc = fma(lds_f64(sdict + 8 * lds_u16(pv + 64 * u)), xv[u], acc);
    return acc;
}
template <class GX>
__device__ __forceinline__ double vi2_row_wide(uint32_t pv, uint32_t pc, uint32_t sdict, const GX& gx, int w) {
    double acc = 0.0;
    for (int t0 = 0; t0 < w; t0 += 8) {
        double xv[8];
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (t0 + u < w) xv[u] = gx(lds_s16(pc + 64 * (t0 + u)));
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (t0 + u < w) acc = fma(lds_f64(sdict + 8 * lds_u16(pv + 64 * (t0 + u))), xv[u], acc);
    }
    return acc;
}

// Packed-word variant (ENC = 1): entry u of a lane is one 32-bit word
// vidx | col16 << 16 at pw + 128 u -- one shared-memory load per entry instead
// of two (half the LSU wavefronts of the index reads).
template <int W, class GX>
__device__ __forceinline__ double vi2_row_w(uint32_t pw, uint32_t sdict, const GX& gx) {
    uint32_t w[W];
#pragma unroll
    for (int u = 0; u < W; ++u) w[u] = lds_u32(pw + 128 * u);
    double xv[W];
#pragma unroll
    for (int u = 0; u < W; ++u) xv[u] = gx((int32_t)w[u] >> 16);
    double acc = 0.0;
#pragma unroll
    for (int u = 0; u < W; ++u) acc = fma(lds_f64(sdict + 8 * (w[u] & 0xffffu)), xv[u], acc);
    return acc;
}
template <class GX>
__device__ __forceinline__ double vi2_row_w_wide(uint32_t pw, uint32_t sdict, const GX& gx, int wd) {
    double acc = 0.0;
    for (int t0 = 0; t0 < wd; t0 += 8) {
        uint32_t w[8];
        double xv[8];
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (t0 + u < wd) w[u] = lds_u32(pw + 128 * (t0 + u));
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (t0 + u < wd) xv[u] = gx((int32_t)w[u] >> 16);
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (t0 + u < wd) acc = fma(lds_f64(sdict + 8 * (w[u] & 0xffffu)), xv[u], acc);
    }
    return acc;
}

// F64 records (ENC = 2): entry u of a lane has its value at pv + 256 u and
// its col16 at pc + 64 u; FMAs in t order (sell_cpt_kernel's arithmetic).
template <int W, class GX>
__device__ __forceinline__ double vi2_row_f(uint32_t pv, uint32_t pc, const GX& gx) {
    double xv[W];
#pragma unroll
    for (int u = 0; u < W; ++u) xv[u] = gx(lds_s16(pc + 64 * u));
    double acc = 0.0;
#pragma unroll
    for (int u = 0; u < W; ++u) acc = fma(lds_f64(pv + 256 * u), xv[u], acc);
    return acc;
}
template <class GX>
__device__ __forceinline__ double vi2_row_f_wide(uint32_t pv, uint32_t pc, const GX& gx, int w) {
    double acc = 0.0;
    for (int t0 = 0; t0 < w; t0 += 8) {
        double xv[8];
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (t0 + u < w) xv[u] = gx(lds_s16(pc + 64 * (t0 + u)));
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (t0 + u < w) acc = fma(lds_f64(pv + 256 * (t0 + u)), xv[u], acc);
    }
    return acc;
}

// The off-band sum of one slot, dispatched on the slice's (warp-uniform) width.
template <int ENC, class GX>
__device__ __forceinline__ double vi2_acc(int w, uint32_t pv, uint32_t pc, uint32_t sdict, const GX& gx) {
    if (ENC == 2) switch (w) {
        case 0: return 0.0;
        case 1: return vi2_row_f<1>(pv, pc, gx);
        case 2: return vi2_row_f<2>(pv, pc, gx);
        case 3: return vi2_row_f<3>(pv, pc, gx);
        case 4: return vi2_row_f<4>(pv, pc, gx);
        case 5: return vi2_row_f<5>(pv, pc, gx);
        case 6: return vi2_row_f<6>(pv, pc, gx);
        case 7: return vi2_row_f<7>(pv, pc, gx);
        case 8: return vi2_row_f<8>(pv, pc, gx);
        default: return vi2_row_f_wide(pv, pc, gx, w);
    }
    if (ENC == 1) switch (w) {
        case 0: return 0.0;
        case 1: return vi2_row_w<1>(pv, sdict, gx);
        case 2: return vi2_row_w<2>(pv, sdict, gx);
        case 3: return vi2_row_w<3>(pv, sdict, gx);
        case 4: return vi2_row_w<4>(pv, sdict, gx);
        case 5: return vi2_row_w<5>(pv, sdict, gx);
        case 6: return vi2_row_w<6>(pv, sdict, gx);
        case 7: return vi2_row_w<7>(pv, sdict, gx);
        case 8: return vi2_row_w<8>(pv, sdict, gx);
        default: return vi2_row_w_wide(pv, sdict, gx, w);
    }
    switch (w) {
        case 0: return 0.0;
        case 1: return vi2_row<1>(pv, pc, sdict, gx);
        case 2: return vi2_row<2>(pv, pc, sdict, gx);
        case 3: return vi2_row<3>(pv, pc, sdict, gx);
        case 4: return vi2_row<4>(pv, pc, sdict, gx);
        case 5: return vi2_row<5>(pv, pc, sdict, gx);
        case 6: return vi2_row<6>(pv, pc, sdict, gx);
        case 7: return vi2_row<7>(pv, pc, sdict, gx);
        case 8: return vi2_row<8>(pv, pc, sdict, gx);
        default: return vi2_row_wide(pv, pc, sdict, gx, w);
    }
}

template <int NCW>
struct Vi2Shape {
    static constexpr int kThreads = 32 * (NCW + 1);
    // 16: 2 x 544 threads (56 regs); 23: 2 x 768 (40 regs); 30: 1 x 992 (64 regs)
    static constexpr int kMinBlocks = NCW == 30 ? 1 : 2;
};

// XW: the x window variant -- each CTA runs a contiguous
// range of tiles and the producer streams the iterate rows those tiles gather
// into a shared-memory ring with the tile records (same mbarriers), so every
// x read of the step is a shared-memory load.  Single-GPU packs only.
template <int NCW, bool BAND, bool REARR, bool CHECK, int ENC, int XWM = 0>
__global__ void __launch_bounds__(Vi2Shape<NCW>::kThreads, XWM ? 1 : Vi2Shape<NCW>::kMinBlocks)
    sell_vi2_kernel(const __grid_constant__ Vi2Args V) {
    constexpr bool XW = XWM != 0;   // 1: mirrored ring, 2: ring with a wrap per entry
    constexpr bool F64 = ENC == 2;
    using R = Vi2Rec<NCW, BAND, REARR, F64>;
    const StepArgs& a = V.a;
    pdl_trigger();
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ uint64_t full[8], empty[8], dbar;
    __shared__ int32_t xoffs[8];   // XW: per stage, ring index of row 0 of its tile's first chunk, minus 256 * chunk
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int S = V.stages;
    unsigned char* stages = smem + V.dict_bytes;
    unsigned char* xring = stages + (size_t)S * V.stage_bytes;
    if (XW) {   // rows the ring has not received (row -1 when xw_off = 0) read as 0
        uint4* z = reinterpret_cast<uint4*>(xring);
        const int nz = (V.xw_rows + 256 * V.xw_mirror) / 2;
        for (int k = threadIdx.x; k < nz; k += blockDim.x) z[k] = make_uint4(0u, 0u, 0u, 0u);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // before the bulk copies overwrite it
    }
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
    const int n_tiles = (int)V.n_tiles;
    // tiles of this CTA: XW a contiguous range [t_begin, t_begin + my_tiles),
    // else c, c + G, c + 2G, ...
    const bool contig = XW || V.contig != 0;
    const int t_begin = contig ? (int)((int64_t)c * n_tiles / G) : c;
    const int t_step = contig ? 1 : G;
    const int my_tiles = contig ? (int)((int64_t)(c + 1) * n_tiles / G) - t_begin
                                : (c < n_tiles ? (n_tiles - 1 - c) / G + 1 : 0);
    const int pro = my_tiles < S ? my_tiles : S;
    if (warp == NCW) {
        // ---------------- producer warp: one bulk copy per tile record ----------------
        // the record offsets of the CTA's next 32 tiles are loaded by the 32
        // lanes together (one round trip per 32 tiles), lane 0 issues
        const uint64_t pol = evict_first_policy();
        if (lane == 0 && V.dict_bytes > 0) {   // dictionary: constant, every CTA reads it (keep it in L2)
            uint64_t keep;
            asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(keep));
            mbar_expect_tx(&dbar, (uint32_t)V.dict_bytes);
            bulk_g2s(smem, V.dict, (uint32_t)V.dict_bytes, &dbar, keep);
        } else if (lane == 0) {
            mbar_arrive(&dbar);   // (F64 records: no dictionary)
        }
        // XW: next iterate chunk to stream (chunks are issued in increasing order)
        int32_t ch_hi = 0, ch_lo = 0;
        int32_t xk = XW && my_tiles > 0 ? __ldg(&V.xw_ch[t_begin].x) : 0;
        const double* xsrc = a.x + a.own_off - V.xw_off;   // 16-B aligned: chunk k starts at xsrc + 256 k
        const int32_t xw_slots = V.xw_rows >> 8;
        // lane 0, before the stage's arrival: where the tile's first chunk sits in the ring
        auto x_base = [&](int st_, int32_t lo) { xoffs[st_] = V.xw_off + (lo % xw_slots - lo) * 256; };
        const int64_t x_avail = V.xw_nx + 1 + V.xw_off;    // rows readable from xsrc (through the sentinel at nx)
        // chunks [xk, hi): runs split at the ring's end, the slots below the
        // mirror copied twice; issue = false only counts the bytes (lane 0)
        auto x_chunks = [&](int32_t hi, uint64_t* bar, bool issue) -> uint32_t {
            uint32_t bytes = 0;
            for (int32_t k = xk; k < hi;) {
                const int32_t slot = k % xw_slots;
                const int32_t run = min(hi - k, xw_slots - slot);
                const int64_t r0 = (int64_t)k * 256, r1 = min((int64_t)(k + run) * 256, x_avail & ~int64_t(1));
                if (r1 > r0) {
                    bytes += (uint32_t)((r1 - r0) * 8);
                    if (issue) bulk_g2s(xring + (size_t)slot * 2048, xsrc + r0, (uint32_t)((r1 - r0) * 8), bar, pol);
                }
                if (slot < V.xw_mirror) {
                    const int64_t m1 = min((int64_t)(k + min(run, V.xw_mirror - slot)) * 256, x_avail & ~int64_t(1));
                    if (m1 > r0) {
                        bytes += (uint32_t)((m1 - r0) * 8);
                        if (issue)
                            bulk_g2s(xring + (size_t)(xw_slots + slot) * 2048, xsrc + r0, (uint32_t)((m1 - r0) * 8),
                                     bar, pol);
                    }
                }
                k += run;
            }
            if (issue) xk = max(xk, hi);
            return bytes;
        };
        auto x_bytes = [&](int32_t hi) -> uint32_t { return x_chunks(hi, nullptr, false); };
        auto x_issue = [&](int32_t hi, uint64_t* bar) { x_chunks(hi, bar, true); };
        int64_t o0 = 0, o1 = 0;
        uint32_t kd = 0;      // fused halo sync: tile kind of the lane's tile
        int32_t chd = 0, chl = 0;   // XW: chunk range of the lane's tile
        int s = 0;
        uint32_t phase = 0;   // parity of the ring pass; reuse i >= S waits for pass (i / S - 1)'s release
        bool waited = false, bad = false;
        int64_t kstep = 0;
        const bool fused = V.hs.on != 0;
        for (int i = 0; i < my_tiles; ++i) {
            const int l = i & 31;
            if (l == 0) {   // offsets of tiles i .. i+31
                const int t = t_begin + (i + lane) * t_step;
                if (i + lane < my_tiles) {
                    o0 = __ldg(V.rec_off + t);
                    o1 = __ldg(V.rec_off + t + 1);
                    kd = fused ? (uint32_t)__ldg(V.hs.tile_kind + t) : 0u;
                    if (XW) {
                        const int2 ch = __ldg(&V.xw_ch[t]);
                        chl = ch.x;
                        chd = ch.y;
                    }
                }
            }
            const int64_t b0 = __shfl_sync(0xffffffffu, o0, l), b1 = __shfl_sync(0xffffffffu, o1, l);
            const uint32_t kind = __shfl_sync(0xffffffffu, kd, l);
            if (XW) {
                ch_hi = __shfl_sync(0xffffffffu, chd, l);
                ch_lo = __shfl_sync(0xffffffffu, chl, l);
            }
            // first tiles were issued before the previous step ended; the stop
            // test comes before any ring reuse: on a stopped launch the
            // consumers release no stage, so waiting on empty[] would hang
            if (i == pro && !waited) {
                pdl_wait();
                waited = true;
                if (a.stop != nullptr && *a.stop) break;
                if (XW) {   // the prologue tiles' iterate chunks (x is the previous step's output)
                    for (int i2 = 0; i2 < pro; ++i2) {
                        const int32_t h2 = __shfl_sync(0xffffffffu, chd, i2), l2 = __shfl_sync(0xffffffffu, chl, i2);
                        if (lane == 0) {
                            x_base(i2, l2);
                            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&full[i2])),
                                         "r"(x_bytes(h2))
                                         : "memory");
                            x_issue(h2, &full[i2]);
                        }
                    }
                }
                if (fused) {   // gated tiles of the prologue: copied, not yet released
                    kstep = *(volatile const int64_t*)V.hs.local;
                    for (int i2 = 0; i2 < pro; ++i2) {
                        const uint32_t k2 = __shfl_sync(0xffffffffu, kd, i2 & 31);
                        if (k2) {
                            hs_gate(V.hs, k2, kstep, bad);
                            if (lane == 0) mbar_arrive(&full[i2]);
                        }
                    }
                }
            }
            if (i >= S) mbar_wait(&empty[s], phase ^ 1u);
            if (lane == 0) {
                const int t = t_begin + i * t_step;
                uint32_t bytes = (uint32_t)(b1 - b0);
                if (XW && i >= pro) {
                    bytes += x_bytes(ch_hi);
                    x_base(s, ch_lo);
                }
                if (V.xpf) {
                    const int64_t r0 = (int64_t)t * NCW * 32, r1 = min(r0 + NCW * 32, a.n_rows);
                    if (r1 > r0) prefetch_l2(a.x + a.own_off + r0, (uint64_t)(r1 - r0) * 8);
                }
                if (kind || (XW && i < pro))   // gated (fused halo sync; XW prologue): the arrival comes later
                    asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&full[s])),
                                 "r"(bytes)
                                 : "memory");
                else
                    mbar_expect_tx(&full[s], bytes);
                bulk_g2s(stages + (size_t)s * V.stage_bytes, V.rec + b0, (uint32_t)(b1 - b0), &full[s], pol);
                if (XW && i >= pro) x_issue(ch_hi, &full[s]);
            }
            if (kind && i >= pro) {
                hs_gate(V.hs, kind, kstep, bad);
                if (lane == 0) mbar_arrive(&full[s]);
            }
            if (++s == S) { s = 0; phase ^= 1u; }
        }
        if (!waited) {
            pdl_wait();
            const bool stopped = a.stop != nullptr && *a.stop;
            if (XW)   // every tile fit the prologue: its chunks now (a stopped launch: release only)
                for (int i2 = 0; i2 < pro; ++i2) {
                    const int32_t h2 = __shfl_sync(0xffffffffu, chd, i2), l2 = __shfl_sync(0xffffffffu, chl, i2);
                    if (lane == 0) {
                        x_base(i2, l2);
                        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&full[i2])),
                                     "r"(stopped ? 0u : x_bytes(h2))
                                     : "memory");
                        if (!stopped) x_issue(h2, &full[i2]);
                    }
                }
            if (fused) {   // every tile fit the prologue: release the gated ones
                kstep = *(volatile const int64_t*)V.hs.local;
                for (int i2 = 0; i2 < pro; ++i2) {
                    const uint32_t k2 = __shfl_sync(0xffffffffu, kd, i2 & 31);
                    if (k2) {
                        if (!stopped) hs_gate(V.hs, k2, kstep, bad);
                        if (lane == 0) mbar_arrive(&full[i2]);
                    }
                }
            }
        } else if ((fused || XW) && a.stop != nullptr && *a.stop) {
            // stopped: the consumers drain the prologue stages; release gated ones
            for (int i2 = 0; i2 < pro; ++i2)
                if ((XW || __shfl_sync(0xffffffffu, kd, i2 & 31)) && lane == 0) mbar_arrive(&full[i2]);
        }
        if (bad && lane == 0) {
            V.hs.ctrl->status = CME_ERR_TIMEOUT;
            V.hs.ctrl->stop = 1;
        }
        if (lane == 0) mbar_wait(&dbar, 0u);   // (no tile may have waited on it)
        if (CHECK) cta_check_partials<NCW + 1, 1>(CheckAcc<1>(), a.partials);
        if (fused) hs_finish(V.hs, G, a.stop);
        return;
    }
    // ---------------- consumer warps: one slice each per tile ----------------
    pdl_wait();
    if (a.stop != nullptr && *a.stop) {
        // the producer saw the same flag; drain the prologue copies before exit
        for (int i = 0; i < pro; ++i) mbar_wait(&full[i], 0u);
        mbar_wait(&dbar, 0u);
        if (CHECK) cta_check_partials<NCW + 1, 1>(CheckAcc<1>(), a.partials);
        if (V.hs.on) hs_finish(V.hs, G, a.stop);
        return;
    }
    const bool fused = V.hs.on != 0;
    const int64_t kstep = fused ? *(volatile const int64_t*)V.hs.local : 0;
    CheckAcc<1> ck;
    {
        const double* xo = a.x + a.own_off;
        double* yo = a.y + a.own_off;
        const bool damp = a.omega != 1.0, unif = a.unif_lam_inv != 0.0;
        const double sc = a.pre_scale != nullptr ? a.pre_scale[0] : 1.0;
        const uint32_t sdict = smem_u32(smem);
        const uint32_t st0 = smem_u32(stages);
        const int n_rows = (int)a.n_rows, slice_end = (int)a.slice_end;
        const uint32_t full0 = smem_u32(full), empty0 = smem_u32(empty);
        const uint32_t sbytes = (uint32_t)V.stage_bytes;
        mbar_wait(&dbar, 0u);
        int s = 0;
        uint32_t phase = 0;
        int q = t_begin * NCW + warp;              // this warp's slice of tile t_begin + i t_step
        const int dq = t_step * NCW;
        const uint32_t sxw = smem_u32(xring);
        uint32_t st = st0;
        for (int i = 0; i < my_tiles; ++i, q += dq) {
            mbar_wait_a(full0 + 8 * s, phase);
            const int32_t xo_t = XW ? xoffs[s] : 0;   // (written by the producer before the stage's arrival)
            const int slot = q * 32 + lane;
            if (q < slice_end && slot < n_rows) {
                const int2 meta = lds_v2(st + 8 * warp);   // {entry offset in the tile, width}
                const int ls = warp * 32 + lane;
                const int r = REARR ? ((slot >> V.win_shift) << V.win_shift) + (int)lds_u8(st + R::kRow + ls) : slot;
                const double* xr = xo + r;
                const uint32_t pv = st + R::kEnt + R::kEntBytes * meta.x + (ENC == 1 ? 4 : ENC == 2 ? 8 : 2) * lane;
                // (ENC 0: the col16 block follows the vidx block; ENC 2: it follows the val_c block)
                const uint32_t pc = F64 ? st + R::kEnt + 10 * meta.x + 256 * meta.y + 2 * lane : pv + 64 * meta.y;
                double acc, x_r, xl = 0.0, xu = 0.0;
                if (XWM == 1) {
                    const GatherS gx{sxw + 8u * (uint32_t)(r + xo_t)};
                    x_r = gx(0);
                    acc = vi2_acc<ENC>(meta.y, pv, pc, sdict, gx);
                    if (BAND) { xl = gx(-1); xu = gx(1); }
                } else if (XWM == 2) {
                    const GatherW gx{sxw + 8u * (uint32_t)(r + xo_t), V.xw_rows - (r + xo_t), 8u * (uint32_t)V.xw_rows};
                    x_r = gx(0);
                    acc = vi2_acc<ENC>(meta.y, pv, pc, sdict, gx);
                    if (BAND) { xl = gx(-1); xu = gx(1); }
                } else {
                    x_r = __ldg(xr);
                    acc = vi2_acc<ENC>(meta.y, pv, pc, sdict, GatherG{xr});
                    if (BAND) { xl = __ldg(xr - 1); xu = __ldg(xr + 1); }
                }
                double sum = acc;
                if (BAND) {
                    const double lo = F64 ? lds_f64(st + R::kLoUp + 8 * ls)
                                          : lds_f64(sdict + 8 * lds_u16(st + R::kLoUp + 2 * ls));
                    const double up = F64 ? lds_f64(st + R::kLoUp + NCW * 256 + 8 * ls)
                                          : lds_f64(sdict + 8 * lds_u16(st + R::kLoUp + NCW * 64 + 2 * ls));
                    sum = fma(lo, xl, up * xu) + acc;
                }
                // F64: the rows are M's (sum = (M x)_r already); inv_d only for checks / transient
                const double id = F64 ? ((CHECK || unif) ? __ldg(a.inv_d + slot) : 1.0) : lds_f64(st + R::kInv + 8 * ls);
                double y = F64 ? (damp ? fma(1.0 - a.omega, x_r, a.omega * sum) : sum)
                               : (damp ? fma(1.0 - a.omega, x_r, a.omega * (id * sum)) : id * sum);
                if (unif) {   // transient: (I + A/Lambda) x with a_rr = -1/id
                    y = F64 ? fma(a.unif_lam_inv, (sum - x_r) / id, x_r) : fma(a.unif_lam_inv, sum - x_r / id, x_r);
                    double* ac = a.acc + a.own_off + r;
                    *ac = fma(a.acc_w, x_r, *ac);
                }
                y *= sc;   // pending 1/sum(y) of the previous check (exact when sc = 1)
                yo[r] = y;
                if (CHECK) ck.add(0, y, x_r * sc, id);
                for (int p = 0; p < a.npush; ++p)   // halo rows straight into the peer's buffer
                    if (r >= a.push_lo[p] && r < a.push_hi[p]) a.push_y[p][r] = y;
            }
            __syncwarp();
            if (lane == 0) {
                if (fused) {
                    const uint32_t kind = __ldg(V.hs.tile_kind + t_begin + i * t_step);
                    if (kind) hs_signal(V.hs, kind, kstep);
                }
                mbar_arrive_a(empty0 + 8 * s);
            }
            st += sbytes;
            if (++s == S) { s = 0; phase ^= 1u; st = st0; }
        }
    }
    if (CHECK) cta_check_partials<NCW + 1, 1>(ck, a.partials);
    if (fused) hs_finish(V.hs, G, a.stop);
}


// ---------------------------------------------------------------------------
// Batched tile records (B = 2, 4, 8 rate sets on one pattern; DESIGN.md
// sec. 9): sell_vib_kernel's arithmetic -- per entry the B-tuple of rates from
// the dictionary (global memory, L1-cached) times the B-wide x gather, FMAs
// in t order per member, row sum times inv_d -- over one contiguous record
// per tile of TS slices:
//   [meta | row8 | loi, upi | inv_d (B per slot, member-minor) | per slice:
//    vidx[32 W], col16[32 W]]
// (the B = 1 record with a B-wide inv_d block), moved by one bulk copy; inv_d
// is read from shared memory.  Single-GPU packs.
template <int TS, int B, bool BAND, bool REARR>
struct Vi2bRec {
    static constexpr int kMeta = ((TS + 1) & ~1) * 8;
    static constexpr int kRow = kMeta;
    static constexpr int kLoUp = kRow + (REARR ? TS * 32 : 0);
    static constexpr int kInv = kLoUp + (BAND ? TS * 128 : 0);
    static constexpr int kEnt = kInv + TS * 256 * B;
};
__host__ __device__ constexpr int vi2b_fixed_bytes(int ts, int b, bool band, bool rearr) {
    return ((ts + 1) & ~1) * 8 + (rearr ? ts * 32 : 0) + (band ? ts * 128 : 0) + ts * 256 * b;
}

template <int NCW, int B>
struct Vi2bShape {
    static constexpr int kThreads = 32 * (NCW + 1);
};

// B-wide tuple read from the shared-memory copy of the dictionary (SD)
template <int B>
__device__ __forceinline__ void lds_tuple(uint32_t a, double* v) {
    if constexpr (B == 2) {
        asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(v[0]), "=d"(v[1]) : "r"(a));
    } else {
#pragma unroll
        for (int b = 0; b < B; ++b) v[b] = lds_f64(a + 8 * b);
    }
}

// SD: the tuple dictionary staged in shared memory (B = 2: 6 318 tuples are
// 101 KB) instead of read through L1, whose pipe the B-wide gathers saturate
template <int NCW, int B, bool BAND, bool REARR, bool CHECK, bool SD = false>
__global__ void __launch_bounds__(Vi2bShape<NCW, B>::kThreads, 1)
    sell_vi2b_kernel(const __grid_constant__ Vi2Args V) {
    using R = Vi2bRec<NCW, B, BAND, REARR>;
    constexpr int U = Chunk<B>::U;   // entries whose loads are in flight together
    const StepArgs& a = V.a;
    pdl_trigger();
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ uint64_t full[8], empty[8], dbar;
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
    const int n_tiles = (int)V.n_tiles;
    const int my_tiles = c < n_tiles ? (n_tiles - 1 - c) / G + 1 : 0;
    const int pro = my_tiles < S ? my_tiles : S;
    unsigned char* stages = smem + (SD ? V.dict_bytes : 0);
    if (warp == NCW) {
        // ---------------- producer warp: one bulk copy per tile record ----------------
        const uint64_t pol = evict_first_policy();
        if (SD && lane == 0) {   // the dictionary: constant, every CTA reads it (keep it in L2)
            uint64_t keep;
            asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(keep));
            mbar_expect_tx(&dbar, (uint32_t)V.dict_bytes);
            bulk_g2s(smem, V.dict, (uint32_t)V.dict_bytes, &dbar, keep);
        }
        int64_t o0 = 0, o1 = 0;
        int s = 0;
        uint32_t phase = 0;
        bool waited = false;
        for (int i = 0; i < my_tiles; ++i) {
            const int l = i & 31;
            if (l == 0 && i + lane < my_tiles) {   // offsets of tiles i .. i+31
                const int t = c + (i + lane) * G;
                o0 = __ldg(V.rec_off + t);
                o1 = __ldg(V.rec_off + t + 1);
            }
            const int64_t b0 = __shfl_sync(0xffffffffu, o0, l), b1 = __shfl_sync(0xffffffffu, o1, l);
            // the first S records were issued before the previous step ended
            // (they are constant); the stop test precedes any ring reuse
            if (i == pro && !waited) {
                pdl_wait();
                waited = true;
                if (a.stop != nullptr && *a.stop) break;
            }
            if (i >= S) mbar_wait(&empty[s], phase ^ 1u);
            if (lane == 0) {
                const uint32_t bytes = (uint32_t)(b1 - b0);
                if (V.xpf) {
                    const int64_t t = c + (int64_t)i * G;
                    const int64_t r0 = t * NCW * 32, r1 = min(r0 + NCW * 32, a.n_rows);
                    if (r1 > r0) prefetch_l2(a.x + (a.own_off + r0) * B, (uint64_t)(r1 - r0) * 8 * B);
                }
                mbar_expect_tx(&full[s], bytes);
                bulk_g2s(stages + (size_t)s * V.stage_bytes, V.rec + b0, bytes, &full[s], pol);
            }
            if (++s == S) { s = 0; phase ^= 1u; }
        }
        if (!waited) pdl_wait();
        if (SD && lane == 0) mbar_wait(&dbar, 0u);   // (no CTA exits with the copy in flight)
        if (CHECK) cta_check_partials<NCW + 1, B>(CheckAcc<B>(), a.partials);
        return;
    }
    // ---------------- consumer warps: one slice each per tile ----------------
    pdl_wait();
    if (a.stop != nullptr && *a.stop) {   // drain the prologue copies before exit
        for (int i = 0; i < pro; ++i) mbar_wait(&full[i], 0u);
        if (CHECK) cta_check_partials<NCW + 1, B>(CheckAcc<B>(), a.partials);
        return;
    }
    CheckAcc<B> ck;
    {
        const double* xo = a.x + a.own_off * B;
        double* yo = a.y + a.own_off * B;
        const double* dict = V.dict;
        const uint32_t sdict = smem_u32(smem);
        if (SD) mbar_wait(&dbar, 0u);
        const int n_rows = (int)a.n_rows, slice_end = (int)a.slice_end;
        const uint32_t full0 = smem_u32(full), empty0 = smem_u32(empty);
        const uint32_t st0 = smem_u32(stages), sbytes = (uint32_t)V.stage_bytes;
        int s = 0;
        uint32_t phase = 0;
        int q = c * NCW + warp;
        const int dq = G * NCW;
        uint32_t st = st0;
        for (int i = 0; i < my_tiles; ++i, q += dq) {
            mbar_wait_a(full0 + 8 * s, phase);
            const int slot = q * 32 + lane;
            if (q < slice_end && slot < n_rows) {
                const int2 meta = lds_v2(st + 8 * warp);   // {entry offset in the tile, width}
                const int ls = warp * 32 + lane;
                const int r = REARR ? ((slot >> V.win_shift) << V.win_shift) + (int)lds_u8(st + R::kRow + ls) : slot;
                RowX<B, BAND> X;
                X.load(xo, r);
                double id[B];
#pragma unroll
                for (int b = 0; b < B; ++b) id[b] = lds_f64(st + R::kInv + 8 * (B * ls + b));
                const uint32_t pv = st + R::kEnt + 4 * meta.x + 2 * lane, pc = pv + 64 * meta.y;
                double acc[B];
#pragma unroll
                for (int b = 0; b < B; ++b) acc[b] = 0.0;
                for (int t0 = 0; t0 < meta.y; t0 += U) {
                    double xv[U][B], vv[U][B];
#pragma unroll
                    for (int u = 0; u < U; ++u)
                        if (t0 + u < meta.y) {
                            ld_vec<B>(xo + (int64_t)(r + lds_s16(pc + 64 * (t0 + u))) * B, xv[u]);
                            if (SD)
                                lds_tuple<B>(sdict + 8 * B * lds_u16(pv + 64 * (t0 + u)), vv[u]);
                            else
                                ld_vec<B>(dict + (int64_t)lds_u16(pv + 64 * (t0 + u)) * B, vv[u]);
                        }
#pragma unroll
                    for (int u = 0; u < U; ++u)
                        if (t0 + u < meta.y)
#pragma unroll
                            for (int b = 0; b < B; ++b) acc[b] = fma(vv[u][b], xv[u][b], acc[b]);
                }
                double lo[B], up[B];
                if (BAND) {
                    if (SD) {
                        lds_tuple<B>(sdict + 8 * B * lds_u16(st + R::kLoUp + 2 * ls), lo);
                        lds_tuple<B>(sdict + 8 * B * lds_u16(st + R::kLoUp + NCW * 64 + 2 * ls), up);
                    } else {
                        ld_vec<B>(dict + (int64_t)lds_u16(st + R::kLoUp + 2 * ls) * B, lo);
                        ld_vec<B>(dict + (int64_t)lds_u16(st + R::kLoUp + NCW * 64 + 2 * ls) * B, up);
                    }
                }
                finish_row_x<B, BAND, CHECK>(a, r, yo, acc, lo, up, id, a.pre_scale, ck, X);
            }
            __syncwarp();
            if (lane == 0) mbar_arrive_a(empty0 + 8 * s);
            st += sbytes;
            if (++s == S) { s = 0; phase ^= 1u; st = st0; }
        }
    }
    if (CHECK) cta_check_partials<NCW + 1, B>(ck, a.partials);
}

}  // namespace cme
