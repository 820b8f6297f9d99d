// refresh.cu — S3 cost refresh (north_star "logistic congestion
// cost, then a warp-shuffle segmented scan into per-layer prefix sums").
//
// The paper only says the wire cost considers wirelength and congestion and defers
// the formula to [3]; our integer reading is R1.
//
// One warp refreshes one 32-position segment of one row (H layers) or column (V
// layers): lane j owns position 32*s + j and all W layer slots of it (one
// 16/32/64-byte sector), computes ec = len + T[clamp(cap - dem)] per slot, runs a
// 5-step __shfl_up_sync inclusive scan per slot, and writes the exclusive
// segment-local prefix P and the segment total ST.  The warp that finishes the
// last dirty segment of a line (per-line atomic counter) rescans that line's
// segment totals into the segment bases SB.  Only segments the previous batch
// committed to are rescanned (byte flags set by the DP's commit), so the bytes
// moved per batch follow the demand that changed, not the grid size.
#include "fgr_internal.cuh"

#include <cstdlib>

template <int W>
struct Vec {
    static __device__ __forceinline__ void load_i32(const int32_t* p, int32_t (&o)[W]) {
#pragma unroll
        for (int q = 0; q < W / 4; q++) {
            int4 t = reinterpret_cast<const int4*>(p)[q];
            o[4 * q] = t.x; o[4 * q + 1] = t.y; o[4 * q + 2] = t.z; o[4 * q + 3] = t.w;
        }
    }
    static __device__ __forceinline__ void load_u32_cg(const uint32_t* p, uint32_t (&o)[W]) {
#pragma unroll
        for (int q = 0; q < W / 4; q++) {
            uint4 t = __ldcg(reinterpret_cast<const uint4*>(p) + q);
            o[4 * q] = t.x; o[4 * q + 1] = t.y; o[4 * q + 2] = t.z; o[4 * q + 3] = t.w;
        }
    }
    static __device__ __forceinline__ void store_u32(uint32_t* p, const uint32_t (&o)[W]) {
#pragma unroll
        for (int q = 0; q < W / 4; q++)
            reinterpret_cast<uint4*>(p)[q] = make_uint4(o[4 * q], o[4 * q + 1], o[4 * q + 2], o[4 * q + 3]);
    }
    static __device__ __forceinline__ void load_u8(const uint8_t* p, uint8_t (&o)[W]) {
        if constexpr (W == 4) {
            uint32_t t = *reinterpret_cast<const uint32_t*>(p);
#pragma unroll
            for (int k = 0; k < 4; k++) o[k] = (uint8_t)(t >> (8 * k));
        } else if constexpr (W == 8) {
            uint2 t = *reinterpret_cast<const uint2*>(p);
#pragma unroll
            for (int k = 0; k < 4; k++) { o[k] = (uint8_t)(t.x >> (8 * k)); o[4 + k] = (uint8_t)(t.y >> (8 * k)); }
        } else {
            uint4 t = *reinterpret_cast<const uint4*>(p);
            uint32_t w4[4] = {t.x, t.y, t.z, t.w};
#pragma unroll
            for (int k = 0; k < 16; k++) o[k] = (uint8_t)(w4[k >> 2] >> (8 * (k & 3)));
        }
    }
};

template <int W>
__device__ __forceinline__ void warp_incl_scan(uint32_t (&x)[W]) {
    const int lane = lane_id();
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
#pragma unroll
        for (int k = 0; k < W; k++) {
            uint32_t t = __shfl_up_sync(0xffffffffu, x[k], off);
            if (lane >= off) x[k] += t;
        }
    }
}

// One segment, transposed: lane = (slot sl = lane % W, run q = lane / W) owns positions
// 32*s + q*W .. + W-1 of one slot.  ec = len + T[clamp(cap - dem)] per position, a serial
// prefix over the run in registers, then an exclusive scan of the run totals across the
// 32/W runs of the slot (log2(32/W) shuffles); P and ST stored.  Same sums as a per-position
// warp scan, a third of the instructions.
template <int W>
struct SegIn {         // one lane's loaded inputs of a segment: demand and capacity of its W positions
    int32_t dem[W];
    uint8_t cap[W];
};

template <int W>
__device__ __forceinline__ void load_segment(const GridView& g, const DirView& d, int line, int s, SegIn<W>& in) {
    const int lane = lane_id();
    const int sl = lane & (W - 1), q = lane / W;
    const int p0 = s * FGR_SEG + q * W;
    const bool slot_ok = sl < d.cnt;
    const size_t base = ((size_t)line * d.len + p0) * W + sl;
#pragma unroll
    for (int j = 0; j < W; j++) {
        const bool ok = slot_ok && p0 + j < d.len - 1;
        in.dem[j] = ok ? d.D[base + (size_t)j * W] : 0;
        in.cap[j] = ok ? d.C[base + (size_t)j * W] : 0;
    }
}

template <int W>
__device__ __forceinline__ void scan_segment(const GridView& g, const DirView& d, int dsel, int line, int s,
                                             const SegIn<W>& in) {
    const int lane = lane_id();
    const int sl = lane & (W - 1), q = lane / W;
    const int p0 = s * FGR_SEG + q * W;
    const bool slot_ok = sl < d.cnt;
    const int span = 2 * g.S + 1;
    const int32_t* tab = g.table + (slot_ok ? g.layer_of_slot[dsel][sl] : 0) * span + g.S;
    const size_t base = ((size_t)line * d.len + p0) * W + sl;
    uint32_t ec[W], run = 0;
#pragma unroll
    for (int j = 0; j < W; j++) {
        uint32_t c = 0;
        if (slot_ok && p0 + j < d.len - 1) {
            int sk = (int)in.cap[j] - in.dem[j];
            sk = sk < -g.S ? -g.S : (sk > g.S ? g.S : sk);
            c = (uint32_t)g.len_cost + (uint32_t)__ldg(tab + sk);
        }
        ec[j] = run;   // exclusive prefix inside the run
        run += c;
    }
    uint32_t x = run;  // inclusive scan of the run totals over the runs of this slot
#pragma unroll
    for (int off = W; off < 32; off <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, off);
        if (lane >= off) x += y;
    }
    const uint32_t before = x - run;
#pragma unroll
    for (int j = 0; j < W; j++)
        if (p0 + j < d.len) d.P[base + (size_t)j * W] = before + ec[j];
    if (q == 32 / W - 1) d.ST[((size_t)line * d.nseg + s) * W + sl] = x;
}

// Segment bases of one line: exclusive scan of all its segment totals.
template <int W>
__device__ __forceinline__ void rebase_line(const DirView& d, int line) {
    const int lane = lane_id();
    uint32_t carry[W];
#pragma unroll
    for (int k = 0; k < W; k++) carry[k] = 0;
    for (int c0 = 0; c0 < d.nseg; c0 += 32) {
        const int s2 = c0 + lane;
        uint32_t v[W], inc[W];
        if (s2 < d.nseg) Vec<W>::load_u32_cg(d.ST + ((size_t)line * d.nseg + s2) * W, v);
        else {
#pragma unroll
            for (int k = 0; k < W; k++) v[k] = 0;
        }
#pragma unroll
        for (int k = 0; k < W; k++) inc[k] = v[k];
        warp_incl_scan<W>(inc);
        if (s2 < d.nseg) {
            uint32_t o[W];
#pragma unroll
            for (int k = 0; k < W; k++) o[k] = carry[k] + inc[k] - v[k];
            Vec<W>::store_u32(d.SB + ((size_t)line * d.nseg + s2) * W, o);
        }
#pragma unroll
        for (int k = 0; k < W; k++) carry[k] += __shfl_sync(0xffffffffu, inc[k], 31);
    }
}

// One task = (line, chunk of 8 segments).  The dirty segments of the chunk are
// rescanned; the warp finishing the last dirty chunk of the line rebuilds the
// segment bases and clears the line's flags.  Returns the segments rescanned.
template <int W, int CS>
__device__ __forceinline__ int refresh_chunk(const GridView& g, const DirView& d, int dsel, int line, int chunk,
                                             bool full) {
    const int lane = lane_id();
    const int lidx = d.line_base + line;
    if (!full && g.dline[lidx] == 0) return 0;
    const uint8_t* f = g.dseg + d.seg_base + (size_t)line * d.nseg;
    const int nchunks = (d.nseg + CS - 1) / CS;
    // dirty chunks of the line (every task of the line computes the same count)
    int nd = 0;
    uint32_t own = 0;
    for (int c0 = 0; c0 < nchunks; c0 += 32) {
        const int c = c0 + lane;
        uint32_t m = 0;
        if (c < nchunks)
            for (int q = 0; q < CS; q++) {
                const int sg = c * CS + q;
                if (sg < d.nseg && (full || f[sg])) m |= 1u << q;
            }
        nd += __popc(__ballot_sync(0xffffffffu, m != 0));
        const uint32_t o = __shfl_sync(0xffffffffu, m, (chunk - c0) & 31);
        if (chunk >= c0 && chunk < c0 + 32) own = o;
    }
    if (own == 0) return 0;
    // two dirty segments in flight: the next segment's loads are issued before this one's scan
    int done = 0;
    int q = __ffs(own) - 1;
    own &= own - 1;
    SegIn<W> cur;
    load_segment<W>(g, d, line, chunk * CS + q, cur);
    for (;;) {
        if (own == 0) {
            scan_segment<W>(g, d, dsel, line, chunk * CS + q, cur);
            done++;
            break;
        }
        const int q2 = __ffs(own) - 1;
        own &= own - 1;
        SegIn<W> nxt;
        load_segment<W>(g, d, line, chunk * CS + q2, nxt);
        scan_segment<W>(g, d, dsel, line, chunk * CS + q, cur);
        done++;
        cur = nxt;
        q = q2;
    }
    // hand-off to the line's last finisher: release this warp's P/ST stores, acquire the others'
    // (acq_rel at GPU scope: the tasks of one line run in different CTAs)
    int last = 0;
    __syncwarp();
    if (lane == 0) {
        unsigned old;
        asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(old) : "l"(&g.linedone[lidx]) : "memory");
        last = (old + 1 == (unsigned)nd);
    }
    last = __shfl_sync(0xffffffffu, last, 0);
    if (last) {
        rebase_line<W>(d, line);
        uint8_t* fw = g.dseg + d.seg_base + (size_t)line * d.nseg;
        for (int sg = lane; sg < d.nseg; sg += 32) fw[sg] = 0;
        if (lane == 0) { g.dline[lidx] = 0; g.linedone[lidx] = 0; }
    }
    return done;
}

template <int WH, int WV, int CS>
__device__ __forceinline__ void refresh_body(const GridView& g, int full) {
    pdl_trigger();   // the next DP kernel may start its prologue now
    pdl_wait();      // the previous batch's commits must be complete
    const int chH = (g.h.nseg + CS - 1) / CS;
    const int chV = (g.v.nseg + CS - 1) / CS;
    const int tH = g.h.lines * chH;
    const int ntasks = tH + g.v.lines * chV;
    const int warp = (int)((blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5);
    const int nwarps = (int)((gridDim.x * (size_t)blockDim.x) >> 5);
    unsigned nh = 0, nv = 0;
    for (int t = warp; t < ntasks; t += nwarps) {
        if (t < tH) {
            const int line = t / chH;
            nh += refresh_chunk<WH, CS>(g, g.h, 0, line, t - line * chH, full);
        } else {
            const int r = t - tH;
            const int line = r / chV;
            nv += refresh_chunk<WV, CS>(g, g.v, 1, line, r - line * chV, full);
        }
    }
    if (lane_id() == 0 && (nh | nv)) {
        atomicAdd(&g.stats[0], (unsigned long long)nh);
        atomicAdd(&g.stats[1], (unsigned long long)nv);
    }
}

template <int WH, int WV>
__global__ void __launch_bounds__(256) k_refresh(GridView g, int full) { refresh_body<WH, WV, FGR_CHUNK_SEGS>(g, full); }

// Launch geometry, fixed by the round-1 A/B measurements: 8 segments per warp task
// (4 / 16: 2.70 / 2.41 ms vs 2.36 ms per t9 step), the compiler's register budget (64 registers, no
// spills; 48 / 40 spill and run slower) and up to 8 CTAs per SM (a single resident wave is slower).
template <int WH, int WV>
static cudaError_t launch_t(fgr_grid* g, cudaStream_t st, bool full, int blocks) {
    const int ps = fgr_prof_begin(g, PROF_REFRESH, st);
    k_refresh<WH, WV><<<blocks, 256, 0, st>>>(g->view, full ? 1 : 0);
    fgr_prof_end(g, ps, st);
    return cudaGetLastError();
}

// One warp per (line, chunk) task; grid capped at 8 CTAs per SM (grid-stride beyond).
// max_tasks (an upper bound on the segments the last batch dirtied) does not size the grid: the
// grid covers every (line, chunk) task and clean lines exit after one flag load, which measured
// faster than a bound-sized grid over a commit-built list.
cudaError_t fgr_launch_refresh_sized(fgr_grid* g, cudaStream_t st, bool full, long long max_tasks) {
    (void)max_tasks;
    const GridView& v = g->view;
    const int cs = FGR_CHUNK_SEGS;
    const long long tasks = (long long)v.h.lines * ((v.h.nseg + cs - 1) / cs) +
                            (long long)v.v.lines * ((v.v.nseg + cs - 1) / cs);
    int blocks = (int)((tasks + 7) / 8);
    const int cap_blocks = g->num_sms * 8;   // grid-stride beyond
    if (blocks > cap_blocks) blocks = cap_blocks;
    if (blocks < 1) blocks = 1;
    g->stats.kernel_launches++;
    const int wh = g->WH, wv = g->WV;
#define FGR_RL(A, B) if (wh == A && wv == B) return launch_t<A, B>(g, st, full, blocks);
    FGR_RL(4, 4) FGR_RL(4, 8) FGR_RL(4, 16) FGR_RL(8, 4) FGR_RL(8, 8) FGR_RL(8, 16) FGR_RL(16, 4) FGR_RL(16, 8)
    FGR_RL(16, 16)
#undef FGR_RL
    return cudaErrorInvalidValue;
}

cudaError_t fgr_launch_refresh(fgr_grid* g, cudaStream_t st, bool full) {
    return fgr_launch_refresh_sized(g, st, full, 0);
}
