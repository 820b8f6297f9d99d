// plan.cu — S0 preprocess, S1 sort, S2 conflict-free batching.
//
// Algorithm 1 repeated until no nets remain (L487-494), over
// nets sorted by ascending bounding-box half-perimeter (L1305-1308, reading R12),
// with "conflict" = the closed bounding boxes share a G-cell (L504, reading R13).
// The repeated greedy passes assign net i (in sorted order) to
//     batch(i) = mex { batch(j) : j before i, box(j) touches box(i) }
// (first fit; proof in DESIGN.md §2).  On the device:
//   1. warp per net: validation, bbox over all nodes (R14), HPWL key, range bound;
//   2. CUB radix sort of (HPWL << 32 | id);
//   3. spatial binning of the sorted boxes into 8x8-cell tiles, (tile, rank) pairs
//      sorted so each tile lists its nets in rank order;
//   4. a persistent ticketed colouring kernel: warps take nets in rank order, scan
//      the tile lists for earlier touching boxes (each pair counted once, in the
//      tile holding the lower-left corner of the intersection), wait for those
//      neighbours' batch ids to be published and take the smallest free id;
//   5. CUB radix sort of (batch << 32 | small-net flag | rank) -> batch CSR.
#include <cub/cub.cuh>

#include "fgr_internal.cuh"

#define TILE_SHIFT 3

namespace {

struct PlanParams {
    int N, nx, ny, L;
    unsigned long long max_ec;   // len_cost + max W
    unsigned long long vmax;     // V(0, L-1)
    int max_nodes_large;         // largest net the CTA path can hold in shared memory
};

__device__ __forceinline__ unsigned long long pack_box(int x0, int y0, int x1, int y1) {
    return (unsigned long long)(uint16_t)x0 | ((unsigned long long)(uint16_t)y0 << 16) |
           ((unsigned long long)(uint16_t)x1 << 32) | ((unsigned long long)(uint16_t)y1 << 48);
}
__device__ __forceinline__ void unpack_box(unsigned long long b, int& x0, int& y0, int& x1, int& y1) {
    x0 = (int)(b & 0xFFFF); y0 = (int)((b >> 16) & 0xFFFF); x1 = (int)((b >> 32) & 0xFFFF); y1 = (int)(b >> 48);
}

// S0 outputs of one net: error flags, the R19 range bound, the (HPWL, id) sort key, the box.
__device__ __forceinline__ void prep_finish(const PlanParams& p, int net, int m, int bad, int x0, int y0, int x1, int y1,
                                            unsigned long long wl, int sb, unsigned long long* keys,
                                            unsigned long long* box, int* msize, int* segb, int* counters) {
    if (bad) {
        atomicMin(&counters[1], net);
        x0 = y0 = x1 = y1 = 0;
    }
    const bool trivial = (m == 1);
    if (trivial) atomicAdd(&counters[0], 1);
    if (!bad && !trivial) {
        // R19: worst case of any route = every unit edge at max cost + every via stack at max
        const unsigned long long bound = wl * p.max_ec + (unsigned long long)(3 * m) * p.vmax;   // Z: 2 bend stacks per edge
        if (bound >= (unsigned long long)FGR_INF || m > p.max_nodes_large) atomicMin(&counters[2], net);
    }
    const unsigned hpwl = trivial ? 0xFFFFu : (unsigned)((x1 - x0) + (y1 - y0));
    keys[net] = ((unsigned long long)hpwl << 32) | (unsigned)net;
    box[net] = pack_box(x0, y0, x1, y1);
    msize[net] = m;
    segb[net] = sb;
}

// S0: one warp per net.
__global__ void k_preprocess(PlanParams p, NetsView nv, unsigned long long* __restrict__ keys,
                             unsigned long long* __restrict__ box, int* __restrict__ msize, int* __restrict__ segb,
                             int* __restrict__ counters /* [0] trivial, [1] err invalid net, [2] err range net */) {
    const int warp = (int)((blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5);
    const int lane = lane_id();
    if (warp >= p.N) return;
    const int net = warp;
    const int a0 = nv.off[net], a1 = nv.off[net + 1];
    const int m = a1 - a0;
    if (m <= 32) return;   // k_preprocess_small
    int bad = (m <= 0);
    int x0 = 0x7FFF, y0 = 0x7FFF, x1 = -1, y1 = -1;
    unsigned long long wl = 0;
    int sb = 0;
    for (int i = lane; i < m; i += 32) {
        const int v = a0 + i;
        const int x = nv.x[v], y = nv.y[v];
        const int lo = nv.plo[v], hi = nv.phi[v];
        if (x < 0 || x >= p.nx || y < 0 || y >= p.ny) bad = 1;
        if (!((lo == -1 && hi == -1) || (lo >= 0 && lo <= hi && hi < p.L))) bad = 1;
        x0 = min(x0, x); y0 = min(y0, y); x1 = max(x1, x); y1 = max(y1, y);
        const int par = nv.par[v];
        if (i == 0) { if (par != -1) bad = 1; }
        else if (par < 0 || par >= i) bad = 1;
        else {
            const int xu = nv.x[a0 + par], yu = nv.y[a0 + par];
            const int dx = abs(x - xu), dy = abs(y - yu);
            if (dx == 0 && dy == 0) bad = 1;   // zero-length tree edge (R8)
            wl += (unsigned long long)(dx + dy);
            sb += (dx >> 5) + (dy >> 5) + 4;
        }
    }
#pragma unroll
    for (int off = 16; off; off >>= 1) {
        bad |= __shfl_xor_sync(0xffffffffu, bad, off);
        x0 = min(x0, __shfl_xor_sync(0xffffffffu, x0, off));
        y0 = min(y0, __shfl_xor_sync(0xffffffffu, y0, off));
        x1 = max(x1, __shfl_xor_sync(0xffffffffu, x1, off));
        y1 = max(y1, __shfl_xor_sync(0xffffffffu, y1, off));
        wl += __shfl_xor_sync(0xffffffffu, wl, off);
        sb += __shfl_xor_sync(0xffffffffu, sb, off);
    }
    if (lane) return;
    prep_finish(p, net, m, bad, x0, y0, x1, y1, wl, sb, keys, box, msize, segb, counters);
}

// S0 for the nets of at most 32 nodes (almost all of them): one thread per net, the same checks
// and outputs as the warp-per-net kernel above (which skips these nets).
__global__ void __launch_bounds__(256) k_preprocess_small(PlanParams p, NetsView nv, unsigned long long* __restrict__ keys,
                                                          unsigned long long* __restrict__ box, int* __restrict__ msize,
                                                          int* __restrict__ segb, int* __restrict__ counters) {
    const int net = (int)(blockIdx.x * (size_t)blockDim.x + threadIdx.x);
    if (net >= p.N) return;
    const int a0 = nv.off[net], a1 = nv.off[net + 1];
    const int m = a1 - a0;
    if (m > 32) return;
    int bad = (m <= 0);
    int x0 = 0x7FFF, y0 = 0x7FFF, x1 = -1, y1 = -1;
    unsigned long long wl = 0;
    int sb = 0;
    for (int i = 0; i < m; i++) {
        const int v = a0 + i;
        const int x = nv.x[v], y = nv.y[v];
        const int lo = nv.plo[v], hi = nv.phi[v];
        if (x < 0 || x >= p.nx || y < 0 || y >= p.ny) bad = 1;
        if (!((lo == -1 && hi == -1) || (lo >= 0 && lo <= hi && hi < p.L))) bad = 1;
        x0 = min(x0, x); y0 = min(y0, y); x1 = max(x1, x); y1 = max(y1, y);
        const int par = nv.par[v];
        if (i == 0) { if (par != -1) bad = 1; }
        else if (par < 0 || par >= i) bad = 1;
        else {
            const int xu = nv.x[a0 + par], yu = nv.y[a0 + par];
            const int dx = abs(x - xu), dy = abs(y - yu);
            if (dx == 0 && dy == 0) bad = 1;   // zero-length tree edge (R8)
            wl += (unsigned long long)(dx + dy);
            sb += (dx >> 5) + (dy >> 5) + 4;
        }
    }
    prep_finish(p, net, m, bad, x0, y0, x1, y1, wl, sb, keys, box, msize, segb, counters);
}

__global__ void k_rank_boxes(int N, const int* __restrict__ counters, const unsigned long long* __restrict__ keys,
                             const unsigned long long* __restrict__ box, unsigned long long* __restrict__ box_r,
                             int* __restrict__ tcount, int tiles_x) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r > N) return;
    const int R = N - counters[0];
    if (r >= R) { tcount[r] = 0; return; }
    const unsigned long long b = box[(unsigned)(keys[r] & 0xFFFFFFFFu)];
    box_r[r] = b;
    int x0, y0, x1, y1;
    unpack_box(b, x0, y0, x1, y1);
    tcount[r] = ((x1 >> TILE_SHIFT) - (x0 >> TILE_SHIFT) + 1) * ((y1 >> TILE_SHIFT) - (y0 >> TILE_SHIFT) + 1);
}

__global__ void k_tile_emit(int R, const unsigned long long* __restrict__ box_r, const int* __restrict__ toff,
                            unsigned long long* __restrict__ tkeys, int tiles_x) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= R) return;
    int x0, y0, x1, y1;
    unpack_box(box_r[r], x0, y0, x1, y1);
    int k = toff[r];
    for (int ty = y0 >> TILE_SHIFT; ty <= (y1 >> TILE_SHIFT); ty++)
        for (int tx = x0 >> TILE_SHIFT; tx <= (x1 >> TILE_SHIFT); tx++)
            tkeys[k++] = ((unsigned long long)(ty * tiles_x + tx) << 32) | (unsigned)r;
}

__global__ void k_tile_bounds(int T, const unsigned long long* __restrict__ tkeys, int* __restrict__ tstart,
                              int* __restrict__ tend, uint4* __restrict__ entries,
                              const unsigned long long* __restrict__ box_r) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= T) return;
    const unsigned long long k = tkeys[i];
    const int t = (int)(k >> 32);
    const unsigned r = (unsigned)(k & 0xFFFFFFFFu);
    const unsigned long long b = box_r[r];
    entries[i] = make_uint4(r, (unsigned)(b & 0xFFFFFFFFu), (unsigned)(b >> 32), 0u);   // rank + its box: one load
    if (i == 0 || (int)(tkeys[i - 1] >> 32) != t) tstart[t] = i;
    if (i == T - 1 || (int)(tkeys[i + 1] >> 32) != t) tend[t] = i + 1;
}

// S2 core: first-fit colouring in rank order, dataflow over published colours.
// A warp scans its net's candidate lists without blocking: colours already
// published are marked at once, unpublished earlier neighbours are deferred and
// waited for only after the whole scan, so the scans of consecutive big nets
// overlap and only the (short) publish chain is serial.
#define COLOR_BITS 1024
#define COLOR_DEFER 128
#define COLOR_UNROLL 8
#define COLOR_CHUNK 16
#define COLOR_BIG_HPWL 24u   // boxes with HPWL >= this take the CTA-per-net phase
__device__ __forceinline__ void mark_colour(uint32_t* bw, int c, int wb) {
    c -= wb;
    if (c >= 0 && c < COLOR_BITS) atomicOr(&bw[c >> 5], 1u << (c & 31));
}

__global__ void __launch_bounds__(256) k_color(int R, const int* __restrict__ rlim, const unsigned long long* __restrict__ box_r,
                                               const int* __restrict__ tstart, const int* __restrict__ tend,
                                               const uint4* __restrict__ entries, int tiles_x, int* color,
                                               int* __restrict__ ticket, int* __restrict__ nbatches,
                                               int* __restrict__ bcount) {
    __shared__ uint32_t bits[8][COLOR_BITS / 32];
    __shared__ int defer[8][COLOR_DEFER];
    __shared__ int ndefer[8];
    // CTA ticket block: base << 32 | next, one 64-bit word so that a rank's (base, index) pair is
    // read atomically (a separate base word could be replaced by a refill between the two reads)
    __shared__ unsigned long long s_tk;
    if (threadIdx.x == 0) s_tk = (unsigned long long)COLOR_CHUNK;   // empty block: first taker refills
    __syncthreads();
    R = *rlim;   // phase 1: the ranks below the big-box threshold (k_color_big does the rest)
    const int w = threadIdx.x >> 5, lane = lane_id();
    uint32_t* bw = bits[w];
    volatile int* vcolor = color;
    for (;;) {
        // Hierarchical tickets: a CTA takes a block of COLOR_CHUNK consecutive ranks with one
        // global atomic; its warps take ranks from it in order through a shared counter.
        // Deadlock-free: the smallest unfinished rank of the earliest unfinished block is
        // always held by a running warp, and every wait is on a smaller rank.
        int r = 0;
        if (lane == 0) {
            for (;;) {
                const unsigned long long tk = atomicAdd(&s_tk, 1ull);
                const int k = (int)(tk & 0xFFFFFFFFull);
                if (k < COLOR_CHUNK) { r = (int)(tk >> 32) + k; break; }
                // block exhausted: one warp refills it; the others spin until the new block is published
                if (k == COLOR_CHUNK) {
                    const int nb = atomicAdd(ticket, COLOR_CHUNK);
                    atomicExch(&s_tk, (unsigned long long)(unsigned)nb << 32);
                } else {
                    while ((int)(*(volatile unsigned long long*)&s_tk & 0xFFFFFFFFull) >= COLOR_CHUNK) __nanosleep(20);
                }
            }
        }
        r = __shfl_sync(0xffffffffu, r, 0);
        if (r >= R) return;
        int x0, y0, x1, y1;
        unpack_box(box_r[r], x0, y0, x1, y1);
        int result = -1;
        for (int wb = 0; result < 0; wb += COLOR_BITS) {
            for (int q = lane; q < COLOR_BITS / 32; q += 32) bw[q] = 0;
            if (lane == 0) ndefer[w] = 0;
            __syncwarp();
            for (int ty = y0 >> TILE_SHIFT; ty <= (y1 >> TILE_SHIFT); ty++)
                for (int tx = x0 >> TILE_SHIFT; tx <= (x1 >> TILE_SHIFT); tx++) {
                    const int t = ty * tiles_x + tx;
                    const int s = tstart[t], e = tend[t];
                    for (int base = s; base < e; base += 32 * COLOR_UNROLL) {
                        int rr[COLOR_UNROLL];
                        unsigned long long bb[COLOR_UNROLL];
#pragma unroll
                        for (int u = 0; u < COLOR_UNROLL; u++) {
                            const int j = base + u * 32 + lane;
                            if (j < e) {
                                const uint4 q = __ldg(entries + j);
                                rr[u] = (int)q.x;
                                bb[u] = (unsigned long long)q.y | ((unsigned long long)q.z << 32);
                            } else {
                                rr[u] = 0x7FFFFFFF;
                                bb[u] = 0ull;
                            }
                        }
                        bool stop = false;
#pragma unroll
                        for (int u = 0; u < COLOR_UNROLL; u++) {
                            stop |= (rr[u] != 0x7FFFFFFF && rr[u] >= r);
                            if (rr[u] < r) {
                                int a0, b0, a1, b1;
                                unpack_box(bb[u], a0, b0, a1, b1);
                                if (!(a1 < x0 || x1 < a0 || b1 < y0 || y1 < b0) &&
                                    (max(a0, x0) >> TILE_SHIFT) == tx && (max(b0, y0) >> TILE_SHIFT) == ty) {
                                    const int c = vcolor[rr[u]];
                                    if (c >= 0) mark_colour(bw, c, wb);
                                    else {
                                        const int k = atomicAdd(&ndefer[w], 1);
                                        if (k < COLOR_DEFER) defer[w][k] = rr[u];
                                        else {
                                            int cc;
                                            while ((cc = vcolor[rr[u]]) < 0) __nanosleep(20);
                                            mark_colour(bw, cc, wb);
                                        }
                                    }
                                }
                            }
                        }
                        if (__any_sync(0xffffffffu, stop)) break;   // lists are rank-sorted
                    }
                }
            __syncwarp();
            const int nd = min(ndefer[w], COLOR_DEFER);
            for (int k = lane; k < nd; k += 32) {
                int cc;
                while ((cc = vcolor[defer[w][k]]) < 0) __nanosleep(20);
                mark_colour(bw, cc, wb);
            }
            __syncwarp();
            // smallest clear bit in this window
            int found = -1;
            for (int q0 = 0; q0 < COLOR_BITS / 32 && found < 0; q0 += 32) {
                const uint32_t word = bw[q0 + lane];
                const uint32_t freeb = ~word;
                const uint32_t any = __ballot_sync(0xffffffffu, freeb != 0);
                if (any) {
                    const int ql = __ffs(any) - 1;
                    const uint32_t fw = __shfl_sync(0xffffffffu, freeb, ql);
                    found = (q0 + ql) * 32 + __ffs(fw) - 1;
                }
            }
            __syncwarp();
            if (found >= 0) result = wb + found;
        }
        if (lane == 0) {
            // the colour word is the only datum a waiting warp reads: publish it without a fence
            atomicExch(&color[r], result);
            atomicMax(nbatches, result + 1);
            atomicAdd(&bcount[result], 1);
        }
    }
}

// First rank whose HPWL reaches `hbig` (keys are sorted by HPWL << 32 | id).
__global__ void k_find_rbig(int R, const unsigned long long* __restrict__ keys_s, unsigned hbig, int* __restrict__ out) {
    int lo = 0, hi = R;
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if ((unsigned)(keys_s[mid] >> 32) < hbig) lo = mid + 1; else hi = mid;
    }
    *out = lo;
}

// Phase 2 of the colouring: ranks with a big box (the tail of the rank order), one CTA
// per net, the 8 warps sharing its tile scan; same first-fit rule and dataflow waits.
#define BIG_DEFER 1024
__global__ void __launch_bounds__(256) k_color_big(int R, const int* __restrict__ rlim,
                                                   const unsigned long long* __restrict__ box_r,
                                                   const int* __restrict__ tstart, const int* __restrict__ tend,
                                                   const uint4* __restrict__ entries, int tiles_x, int* color,
                                                   int* __restrict__ ticket, int* __restrict__ nbatches,
                                                   int* __restrict__ bcount) {
    __shared__ uint32_t bits[COLOR_BITS / 32];
    __shared__ int defer[BIG_DEFER];
    __shared__ int ndefer, s_r, s_res;
    const int w = threadIdx.x >> 5, lane = lane_id(), tid = threadIdx.x;
    volatile int* vcolor = color;
    const int R0 = *rlim;
    for (;;) {
        if (tid == 0) s_r = R0 + atomicAdd(ticket, 1);
        __syncthreads();
        const int r = s_r;
        if (r >= R) return;
        int x0, y0, x1, y1;
        unpack_box(box_r[r], x0, y0, x1, y1);
        const int tx0 = x0 >> TILE_SHIFT, ty0 = y0 >> TILE_SHIFT;
        const int ntx = (x1 >> TILE_SHIFT) - tx0 + 1, nty = (y1 >> TILE_SHIFT) - ty0 + 1;
        int result = -1;
        for (int wb = 0; result < 0; wb += COLOR_BITS) {
            if (tid < COLOR_BITS / 32) bits[tid] = 0;
            if (tid == 0) { ndefer = 0; s_res = -1; }
            __syncthreads();
            for (int ti = w; ti < ntx * nty; ti += 8) {
                const int tx = tx0 + ti % ntx, ty = ty0 + ti / ntx;
                const int t = ty * tiles_x + tx;
                const int s = tstart[t], e = tend[t];
                for (int base = s; base < e; base += 32 * COLOR_UNROLL) {
                    int rr[COLOR_UNROLL];
                    unsigned long long bb[COLOR_UNROLL];
#pragma unroll
                    for (int u = 0; u < COLOR_UNROLL; u++) {
                        const int j = base + u * 32 + lane;
                        if (j < e) {
                            const uint4 q = __ldg(entries + j);
                            rr[u] = (int)q.x;
                            bb[u] = (unsigned long long)q.y | ((unsigned long long)q.z << 32);
                        } else {
                            rr[u] = 0x7FFFFFFF;
                            bb[u] = 0ull;
                        }
                    }
                    bool stop = false;
#pragma unroll
                    for (int u = 0; u < COLOR_UNROLL; u++) {
                        stop |= (rr[u] != 0x7FFFFFFF && rr[u] >= r);
                        if (rr[u] < r) {
                            int a0, b0, a1, b1;
                            unpack_box(bb[u], a0, b0, a1, b1);
                            if (!(a1 < x0 || x1 < a0 || b1 < y0 || y1 < b0) &&
                                (max(a0, x0) >> TILE_SHIFT) == tx && (max(b0, y0) >> TILE_SHIFT) == ty) {
                                const int c = vcolor[rr[u]];
                                if (c >= 0) mark_colour(bits, c, wb);
                                else {
                                    const int k = atomicAdd(&ndefer, 1);
                                    if (k < BIG_DEFER) defer[k] = rr[u];
                                    else {
                                        int cc;
                                        while ((cc = vcolor[rr[u]]) < 0) __nanosleep(20);
                                        mark_colour(bits, cc, wb);
                                    }
                                }
                            }
                        }
                    }
                    if (__any_sync(0xffffffffu, stop)) break;
                }
            }
            __syncthreads();
            const int nd = min(ndefer, BIG_DEFER);
            for (int k = tid; k < nd; k += blockDim.x) {
                int cc;
                while ((cc = vcolor[defer[k]]) < 0) __nanosleep(20);
                mark_colour(bits, cc, wb);
            }
            __syncthreads();
            if (w == 0) {
                const uint32_t freeb = ~bits[lane];
                const uint32_t any = __ballot_sync(0xffffffffu, freeb != 0);
                if (any && lane == 0) {
                    const int ql = __ffs(any) - 1;
                    const uint32_t fw = ~bits[ql];
                    s_res = ql * 32 + __ffs(fw) - 1;
                }
            }
            __syncthreads();
            if (s_res >= 0) result = wb + s_res;
            __syncthreads();
        }
        if (tid == 0) {
            atomicExch(&color[r], result);
            atomicMax(nbatches, result + 1);
            atomicAdd(&bcount[result], 1);
        }
        __syncthreads();
    }
}

// batch-major, then larger nets first (large nets lead each batch; similar sizes share a warp), then rank
__global__ void k_batch_keys(int R, const int* __restrict__ color, const unsigned long long* __restrict__ keys,
                             const int* __restrict__ msize, unsigned long long* __restrict__ bkeys) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= R) return;
    const int id = (int)(keys[r] & 0xFFFFFFFFu);
    const unsigned inv = 2047u - (unsigned)min(msize[id], 2047);
    bkeys[r] = ((unsigned long long)color[r] << 42) | ((unsigned long long)inv << 31) | (unsigned)r;
}

__global__ void k_finalize(int N, const int* __restrict__ counters, const unsigned long long* __restrict__ keys,
                           const unsigned long long* __restrict__ bkeys, const int* __restrict__ msize,
                           const int* __restrict__ segb, int* __restrict__ order, int* __restrict__ batch_of_net,
                           int* __restrict__ nlarge, int* __restrict__ maxm, unsigned long long* __restrict__ segsum,
                           int* __restrict__ ntwo, int* __restrict__ n9, int* __restrict__ lsplit, int lim) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= N) return;
    const int R = N - counters[0];
    if (i < R) {
        const unsigned long long bk = bkeys[i];
        const int r = (int)(bk & 0x7FFFFFFFu);
        const int c = (int)(bk >> 42);
        const int id = (int)(keys[r] & 0xFFFFFFFFu);
        order[i] = id;
        batch_of_net[id] = c;
        const int m = msize[id];
        if (m > FGR_SMALL_NET) {
            atomicAdd(&nlarge[c], 1);
            atomicMax(&maxm[c], m);
            // large-net size buckets (> fgr_top_limit, 512, 256, 128, 64)
            if (m > 64) atomicAdd(&lsplit[5 * c + 4], 1);
            if (m > 128) atomicAdd(&lsplit[5 * c + 3], 1);
            if (m > 256) atomicAdd(&lsplit[5 * c + 2], 1);
            if (m > 512) atomicAdd(&lsplit[5 * c + 1], 1);
            if (m > lim) atomicAdd(&lsplit[5 * c + 0], 1);
        }
        // per-batch sum of dirty-segment bounds (refresh launch sizing); keys are
        // batch-sorted, so a warp almost always shares one batch id
        const unsigned long long v = (unsigned long long)segb[id];
        const unsigned act = __activemask();
        const int lead = __ffs(act) - 1;
        const int c0 = __shfl_sync(act, c, lead);
        if (__all_sync(act, c == c0)) {
            const unsigned sum = __reduce_add_sync(act, (unsigned)v);
            const unsigned two = __reduce_add_sync(act, m == 2 ? 1u : 0u);
            const unsigned nine = __reduce_add_sync(act, (m > FGR_MID_NET && m <= FGR_SMALL_NET) ? 1u : 0u);
            if (lane_id() == lead) {
                atomicAdd(&segsum[c], (unsigned long long)sum);
                if (two) atomicAdd(&ntwo[c], (int)two);
                if (nine) atomicAdd(&n9[c], (int)nine);
            }
        } else {
            atomicAdd(&segsum[c], v);
            if (m == 2) atomicAdd(&ntwo[c], 1);
            if (m > FGR_MID_NET && m <= FGR_SMALL_NET) atomicAdd(&n9[c], 1);
        }
    } else {
        const int id = (int)(keys[i] & 0xFFFFFFFFu);
        order[i] = id;
        batch_of_net[id] = -1;
    }
}

template <typename T>
T* take(fgr_grid* g, int slot, size_t n, cudaError_t* e) {
    return (T*)fgr_scratch(g->s_plan[slot], n * sizeof(T), e);
}

int bits_for(long long v) {
    int b = 1;
    while ((1LL << b) <= v) b++;
    return b;
}

}  // namespace

// largest net the CTA path can hold (shared memory), capped by its depth arrays
static int max_large_nodes(const fgr_grid*) {
    return 65535;   // net-local uint16 indices; nets above fgr_large_limit take k_dp_hld (global workspace)
}

extern "C" FGR_API fgr_status fgr_plan(fgr_grid* g, const fgr_nets* nets, int32_t* batch_of_net, int32_t* order,
                                       int32_t* batch_offset, int32_t* num_batches, void* stream) {
    if (!g || !nets || !num_batches) return fgr_set_error(FGR_ERR_INVALID, "NULL argument");
    if (g->broken) return fgr_set_error(FGR_ERR_STATE, "grid unusable after an earlier CUDA/NCCL error");
    const int N = nets->num_nets;
    if (N < 0 || nets->num_nodes < 0) return fgr_set_error(FGR_ERR_INVALID, "negative sizes");
    if (N > 0 && (!nets->node_offset || !nets->x || !nets->y || !nets->pin_lo || !nets->pin_hi || !nets->parent ||
                  !batch_of_net || !order || !batch_offset))
        return fgr_set_error(FGR_ERR_INVALID, "NULL array");
    cudaStream_t st = (cudaStream_t)stream;
    FGR_CHECK_CUDA(g, cudaSetDevice(g->device));
    g->cache.valid = false;
    *num_batches = 0;
    if (N == 0) {
        FGR_CHECK_CUDA(g, cudaMemsetAsync(batch_offset, 0, sizeof(int32_t), st));
        FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));
        g->cache.valid = true;
        g->cache.prep_valid = false;
        g->hy.cached = false;
        g->cache.exec = order;
        g->cache.nets = *nets; g->cache.order = order; g->cache.batch_offset = batch_offset; g->cache.num_batches = 0;
        return FGR_OK;
    }
    cudaError_t e = cudaSuccess;
    const NetsView nv = fgr_nets_view(nets);
    PlanParams p;
    p.N = N; p.nx = g->nx; p.ny = g->ny; p.L = g->L;
    int maxw = 0;
    for (int l = 0; l < g->L; l++) maxw = g->ovf_weight[l] > maxw ? g->ovf_weight[l] : maxw;
    p.max_ec = (unsigned long long)g->len_cost + (unsigned long long)maxw;
    p.vmax = g->view.viapre[g->L - 1];
    p.max_nodes_large = max_large_nodes(g);

    const int tiles_x = ((g->nx - 1) >> TILE_SHIFT) + 1, tiles_y = ((g->ny - 1) >> TILE_SHIFT) + 1;
    const int ntiles = tiles_x * tiles_y;
    auto* keys = take<unsigned long long>(g, 0, N, &e);
    auto* keys_s = take<unsigned long long>(g, 1, N, &e);
    auto* box = take<unsigned long long>(g, 2, N, &e);
    auto* box_r = take<unsigned long long>(g, 3, (size_t)N + 1, &e);
    auto* msize = take<int>(g, 4, N, &e);
    auto* segb = take<int>(g, 5, N, &e);
    auto* tcount = take<int>(g, 6, (size_t)N + 1, &e);
    // counters: [0] trivial [1] err invalid [2] err range [3] ticket [4] nbatches [5..] spare
    auto* counters = take<int>(g, 7, 16 + 2 * (size_t)ntiles, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "plan scratch");
    int* tstart = counters + 16;
    int* tend = tstart + ntiles;
    int hc[8] = {0, 0x7FFFFFFF, 0x7FFFFFFF, 0, 0, 0, 0, 0};
    FGR_CHECK_CUDA(g, cudaMemcpyAsync(counters, hc, sizeof(hc), cudaMemcpyHostToDevice, st));
    FGR_CHECK_CUDA(g, cudaMemsetAsync(tstart, 0, 2 * sizeof(int) * ntiles, st));
    int ps = fgr_prof_begin(g, PROF_PRE, st);
    k_preprocess_small<<<(unsigned)(((size_t)N + 255) / 256), 256, 0, st>>>(p, nv, keys, box, msize, segb, counters);
    k_preprocess<<<(unsigned)(((size_t)N * 32 + 255) / 256), 256, 0, st>>>(p, nv, keys, box, msize, segb, counters);
    fgr_prof_end(g, ps, st);
    FGR_CHECK_CUDA(g, cudaGetLastError());
    // S1: sort by (HPWL, id)
    size_t tmp_bytes = 0;
    cub::DeviceRadixSort::SortKeys(nullptr, tmp_bytes, keys, keys_s, N, 0, 48, st);
    void* tmp = fgr_scratch(g->s_plan[8], tmp_bytes, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "plan sort scratch");
    ps = fgr_prof_begin(g, PROF_SORT, st);
    FGR_CHECK_CUDA(g, cub::DeviceRadixSort::SortKeys(tmp, tmp_bytes, keys, keys_s, N, 0, 48, st));
    fgr_prof_end(g, ps, st);
    k_rank_boxes<<<(N + 1 + 255) / 256, 256, 0, st>>>(N, counters, keys_s, box, box_r, tcount, tiles_x);
    FGR_CHECK_CUDA(g, cudaGetLastError());
    // tile offsets
    int* toff = (int*)keys;   // keys (N x 8 B) are no longer needed: reuse as N+1 ints
    tmp_bytes = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, tcount, toff, N + 1, st);
    tmp = fgr_scratch(g->s_plan[8], tmp_bytes, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "plan scan scratch");
    FGR_CHECK_CUDA(g, cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, tcount, toff, N + 1, st));
    int hbuf[4];
    FGR_CHECK_CUDA(g, cudaMemcpyAsync(hbuf, counters, 3 * sizeof(int), cudaMemcpyDeviceToHost, st));
    int T = 0;
    FGR_CHECK_CUDA(g, cudaMemcpyAsync(&T, toff + N, sizeof(int), cudaMemcpyDeviceToHost, st));
    FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));  // sync 1 of 2
    if (hbuf[1] != 0x7FFFFFFF)
        return fgr_set_error(FGR_ERR_INVALID, "net %d is malformed (node count, coordinates, pin span, parent "
                             "index (must be in [0, j-1]) or a zero-length tree edge)", hbuf[1]);
    if (hbuf[2] != 0x7FFFFFFF)
        return fgr_set_error(FGR_ERR_RANGE, "net %d: worst-case cost may reach 2^31 or it has more than %d nodes",
                             hbuf[2], p.max_nodes_large);
    const int R = N - hbuf[0];
    // S2: binning
    auto* tkeys = take<unsigned long long>(g, 9, (size_t)T + 1, &e);
    auto* tkeys_s = take<unsigned long long>(g, 10, (size_t)T + 1, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "plan tile scratch");
    uint4* entries = take<uint4>(g, 12, (size_t)T + 1, &e);   // (rank, box) per tile entry
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "plan tile entries");
    int* color = tcount;          // N+1 ints, tcount no longer needed after the scan
    if (R > 0) {
        k_tile_emit<<<(R + 255) / 256, 256, 0, st>>>(R, box_r, toff, tkeys, tiles_x);
        FGR_CHECK_CUDA(g, cudaGetLastError());
        tmp_bytes = 0;
        const int tb = 32 + bits_for(ntiles);
        cub::DeviceRadixSort::SortKeys(nullptr, tmp_bytes, tkeys, tkeys_s, T, 0, tb, st);
        tmp = fgr_scratch(g->s_plan[8], tmp_bytes, &e);
        if (e != cudaSuccess) return fgr_cuda_fail(g, e, "plan tile sort scratch");
        ps = fgr_prof_begin(g, PROF_SORT, st);
        FGR_CHECK_CUDA(g, cub::DeviceRadixSort::SortKeys(tmp, tmp_bytes, tkeys, tkeys_s, T, 0, tb, st));
        fgr_prof_end(g, ps, st);
        k_tile_bounds<<<(T + 255) / 256, 256, 0, st>>>(T, tkeys_s, tstart, tend, entries, box_r);
        FGR_CHECK_CUDA(g, cudaGetLastError());
    }
    // colouring
    auto* bc = take<int>(g, 11, 10 * ((size_t)R + 1), &e);   // bcount | nlarge | maxm | ntwo | n9 | lsplit[5]
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "plan batch scratch");
    int* d_bcount = bc;
    int* d_nlarge = bc + (R + 1);
    int* d_maxm = bc + 2 * (R + 1);
    int* d_ntwo = bc + 3 * (R + 1);
    int* d_n9 = bc + 4 * (R + 1);
    int* d_ls = bc + 5 * (R + 1);
    FGR_CHECK_CUDA(g, cudaMemsetAsync(bc, 0, 10 * sizeof(int) * ((size_t)R + 1), st));
    FGR_CHECK_CUDA(g, cudaMemsetAsync(color, 0xFF, sizeof(int) * ((size_t)N + 1), st));
    FGR_CHECK_CUDA(g, cudaMemsetAsync(batch_of_net, 0xFF, sizeof(int) * (size_t)N, st));
    if (R > 0) {
        int occ = 1;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_color, 256, 0);
        int blocks = g->num_sms * (occ > 0 ? occ : 1);
        int need = (R + 7) / 8;
        if (blocks > need) blocks = need;
        ps = fgr_prof_begin(g, PROF_COLOR, st);
        // ranks below the big-box threshold: a warp per net; the big boxes: a CTA per net
        k_find_rbig<<<1, 1, 0, st>>>(R, keys_s, COLOR_BIG_HPWL, counters + 5);
        k_color<<<blocks, 256, 0, st>>>(R, counters + 5, box_r, tstart, tend, entries, tiles_x, color, counters + 3,
                                        counters + 4, d_bcount);
        k_color_big<<<g->num_sms * 4, 256, 0, st>>>(R, counters + 5, box_r, tstart, tend, entries, tiles_x, color,
                                                   counters + 6, counters + 4, d_bcount);
        fgr_prof_end(g, ps, st);
        FGR_CHECK_CUDA(g, cudaGetLastError());
        g->stats.kernel_launches++;
    }
    // batch CSR
    auto* bkeys = (unsigned long long*)box;      // box (N x 8 B) no longer needed
    auto* bkeys_s = keys;                        // keys region (toff) no longer needed after emit
    if (R > 0) {
        k_batch_keys<<<(R + 255) / 256, 256, 0, st>>>(R, color, keys_s, msize, bkeys);
        FGR_CHECK_CUDA(g, cudaGetLastError());
        tmp_bytes = 0;
        const int bb = 42 + bits_for(R);
        cub::DeviceRadixSort::SortKeys(nullptr, tmp_bytes, bkeys, bkeys_s, R, 0, bb, st);
        tmp = fgr_scratch(g->s_plan[8], tmp_bytes, &e);
        if (e != cudaSuccess) return fgr_cuda_fail(g, e, "plan batch sort scratch");
        ps = fgr_prof_begin(g, PROF_SORT, st);
        FGR_CHECK_CUDA(g, cub::DeviceRadixSort::SortKeys(tmp, tmp_bytes, bkeys, bkeys_s, R, 0, bb, st));
        fgr_prof_end(g, ps, st);
    }
    tmp_bytes = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, d_bcount, batch_offset, R + 1, st);
    tmp = fgr_scratch(g->s_plan[8], tmp_bytes, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "plan offset scratch");
    FGR_CHECK_CUDA(g, cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, d_bcount, batch_offset, R + 1, st));
    auto* segsum = (unsigned long long*)box_r;   // box_r no longer needed after colouring
    FGR_CHECK_CUDA(g, cudaMemsetAsync(segsum, 0, sizeof(unsigned long long) * ((size_t)R + 1), st));
    k_finalize<<<(N + 255) / 256, 256, 0, st>>>(N, counters, keys_s, bkeys_s, msize, segb, order, batch_of_net,
                                                d_nlarge, d_maxm, segsum, d_ntwo, d_n9, d_ls, fgr_top_limit(g));
    FGR_CHECK_CUDA(g, cudaGetLastError());
    g->stats.kernel_launches += 7;
    int B = 0;
    FGR_CHECK_CUDA(g, cudaMemcpyAsync(&B, counters + 4, sizeof(int), cudaMemcpyDeviceToHost, st));
    FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));  // sync 2 of 2
    PlanCache& c = g->cache;
    FGR_CHECK_CUDA(g, fgr_mirrors_reserve(c, B));
    if (B > 0) {   // pinned mirrors: the copies are queued, one synchronisation
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_off, batch_offset, sizeof(int) * (B + 1), cudaMemcpyDeviceToHost, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_nlarge, d_nlarge, sizeof(int) * B, cudaMemcpyDeviceToHost, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_maxm, d_maxm, sizeof(int) * B, cudaMemcpyDeviceToHost, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_ntwo, d_ntwo, sizeof(int) * B, cudaMemcpyDeviceToHost, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_n9, d_n9, sizeof(int) * B, cudaMemcpyDeviceToHost, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_lsplit, d_ls, sizeof(int) * 5 * B, cudaMemcpyDeviceToHost, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_segb, segsum, sizeof(long long) * B, cudaMemcpyDeviceToHost, st));
        FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));
    }
    c.valid = true;
    c.prep_valid = false;
    g->hy.cached = false;
    c.exec = order;
    c.nets = *nets;
    c.order = order;
    c.batch_offset = batch_offset;
    c.num_batches = B;
    *num_batches = B;
    return FGR_OK;
}
