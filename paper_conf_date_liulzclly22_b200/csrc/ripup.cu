// ripup.cu — rip-up set extraction and the ordered task graph.
//
// After the pattern-routing stage, "we first extract the nets to rip up" (PAPER.md
// L398-402): the nets whose committed routes use an overflowed wire edge (demand >
// capacity, reading R26) are rerouted (L1109-1115).  Those routing tasks are then
// ordered by the task graph scheduler (§III-B): conflict = closed boxes
// share a G-cell (R13), task IDs = the (HPWL, id) sort, one root batch by one pass
// of Algorithm 1, every conflicting pair ordered root -> non-root, else from the
// smaller task ID to the larger (reading R27).
//
// Kernels:
//   k_ovf_totals  grid-stride stream over the demand and capacity arrays (int4 + uchar4
//                 per thread, HBM-bound): overflowed wire edges and total overflow;
//   k_ovf_nets    one warp per net: each lane walks the unit edges of its nodes' legs;
//   task graph    tile lists of the task boxes (each conflicting pair found once per
//                 task, in the tile holding the lower-left corner of the intersection),
//                 the root batch as a rank-order dataflow (a task is a root iff no earlier
//                 neighbour is; a warp waits only on smaller ranks held by running warps),
//                 then the oriented edges sorted into a CSR.
#include <cub/cub.cuh>

#include <algorithm>

#include "fgr_internal.cuh"

namespace {

constexpr int kTileShift = 5;   // 32 x 32 G-cell tiles for the conflict search

__global__ void k_ovf_totals(DirView d, unsigned long long* __restrict__ out) {
    const long long n4 = (long long)d.lines * d.len * d.W / 4;
    unsigned long long cnt = 0, sum = 0;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n4; i += (long long)gridDim.x * blockDim.x) {
        const long long e0 = 4 * i;
        const long long pos = e0 / d.W;             // W is a power of two >= 4: one position per int4
        const int slot0 = (int)(e0 % d.W);
        if ((int)(pos % d.len) == d.len - 1 || slot0 >= d.cnt) continue;   // no wire edge / padding
        const int4 dv = reinterpret_cast<const int4*>(d.D)[i];
        const uchar4 cv = reinterpret_cast<const uchar4*>(d.C)[i];
        const int dd[4] = {dv.x, dv.y, dv.z, dv.w};
        const int cc[4] = {cv.x, cv.y, cv.z, cv.w};
#pragma unroll
        for (int k = 0; k < 4; k++)
            if (slot0 + k < d.cnt && dd[k] > cc[k]) { cnt++; sum += (unsigned long long)(dd[k] - cc[k]); }
    }
    cnt = __reduce_add_sync(0xffffffffu, (unsigned)cnt);
#pragma unroll
    for (int off = 16; off; off >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, off);
    if (lane_id() == 0 && (cnt || sum)) { atomicAdd(&out[0], cnt); atomicAdd(&out[1], sum); }
}

__device__ __forceinline__ bool leg_over(const DirView& d, int line, int a, int b, int sl) {
    const int lo = min(a, b), hi = max(a, b);
    const size_t base = (size_t)line * d.len;
    for (int p = lo; p < hi; p++) {
        const size_t e = (base + p) * d.W + sl;
        if (d.D[e] > (int)d.C[e]) return true;
    }
    return false;
}

// one warp per net: violating[net] = some unit edge of a committed leg is overflowed
__global__ void k_ovf_nets(GridView g, NetsView nv, int N, const uint32_t* __restrict__ seg,
                           const int32_t* __restrict__ zmid, uint8_t* __restrict__ viol) {
    const int net = (int)((blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5);
    if (net >= N) return;
    const int a0 = nv.off[net], m = nv.off[net + 1] - a0;
    bool bad = false;
    for (int i = 1 + lane_id(); i < m && !bad; i += 32) {
        const int v = a0 + i, u = a0 + nv.par[v];
        const int xv = nv.x[v], yv = nv.y[v], xu = nv.x[u], yu = nv.y[u];
        const uint32_t s = seg[v];
        const int bend = s & 0xFF, ls = (s >> 8) & 0xFF, lt = (s >> 16) & 0xFF, straight = (s >> 24) & 0xFF;
        const int sls = g.slot[ls], slt = g.slot[lt];
        if (straight) {
            bad = yv == yu ? leg_over(g.h, yv, xv, xu, slt) : leg_over(g.v, xv, yv, yu, slt);
        } else if (bend >= 2) {
            const uint32_t z = (uint32_t)zmid[v];
            const int mid = (int)(z & 0xFFFF), slb = g.slot[(z >> 16) & 0xFF];
            if (bend == 2)
                bad = leg_over(g.h, yv, xv, mid, sls) || leg_over(g.v, mid, yv, yu, slb) || leg_over(g.h, yu, mid, xu, slt);
            else
                bad = leg_over(g.v, xv, yv, mid, sls) || leg_over(g.h, mid, xv, xu, slb) || leg_over(g.v, xu, mid, yu, slt);
        } else if (bend == 0) {
            bad = leg_over(g.h, yv, xv, xu, sls) || leg_over(g.v, xu, yv, yu, slt);
        } else {
            bad = leg_over(g.v, xv, yv, yu, sls) || leg_over(g.h, yu, xv, xu, slt);
        }
    }
    bad = __any_sync(0xffffffffu, bad);
    if (lane_id() == 0) viol[net] = bad ? 1 : 0;
}

// ---------------------------------------------------------------- task graph
struct Box { int x0, y0, x1, y1; };

// one warp per task: (HPWL << 32 | net id) key, box over all tree nodes (R14)
__global__ void k_tg_keys(int R, const int32_t* __restrict__ tasks, NetsView nv, unsigned long long* __restrict__ keys) {
    const int r = (int)((blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5);
    if (r >= R) return;
    const int net = tasks[r];
    const int a0 = nv.off[net], m = nv.off[net + 1] - a0;
    int x0 = 0x7FFF, y0 = 0x7FFF, x1 = -1, y1 = -1;
    for (int i = lane_id(); i < m; i += 32) {
        x0 = min(x0, (int)nv.x[a0 + i]); x1 = max(x1, (int)nv.x[a0 + i]);
        y0 = min(y0, (int)nv.y[a0 + i]); y1 = max(y1, (int)nv.y[a0 + i]);
    }
    x0 = __reduce_min_sync(0xffffffffu, x0); y0 = __reduce_min_sync(0xffffffffu, y0);
    x1 = __reduce_max_sync(0xffffffffu, x1); y1 = __reduce_max_sync(0xffffffffu, y1);
    if (lane_id() == 0) keys[r] = ((unsigned long long)((x1 - x0) + (y1 - y0)) << 32) | (unsigned)net;
}

__global__ void k_tg_boxes(int R, const unsigned long long* __restrict__ keys_s, NetsView nv, int32_t* __restrict__ order,
                           Box* __restrict__ box, int32_t* __restrict__ ntile) {
    const int r = (int)((blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5);
    if (r >= R) return;
    const int net = (int)(keys_s[r] & 0xFFFFFFFFull);
    const int a0 = nv.off[net], m = nv.off[net + 1] - a0;
    int x0 = 0x7FFF, y0 = 0x7FFF, x1 = -1, y1 = -1;
    for (int i = lane_id(); i < m; i += 32) {
        x0 = min(x0, (int)nv.x[a0 + i]); x1 = max(x1, (int)nv.x[a0 + i]);
        y0 = min(y0, (int)nv.y[a0 + i]); y1 = max(y1, (int)nv.y[a0 + i]);
    }
    x0 = __reduce_min_sync(0xffffffffu, x0); y0 = __reduce_min_sync(0xffffffffu, y0);
    x1 = __reduce_max_sync(0xffffffffu, x1); y1 = __reduce_max_sync(0xffffffffu, y1);
    if (lane_id() == 0) {
        order[r] = net;
        box[r] = Box{x0, y0, x1, y1};
        ntile[r] = ((x1 >> kTileShift) - (x0 >> kTileShift) + 1) * ((y1 >> kTileShift) - (y0 >> kTileShift) + 1);
    }
}

__global__ void k_tg_tile_emit(int R, const Box* __restrict__ box, const int32_t* __restrict__ toff, int tiles_x,
                               unsigned long long* __restrict__ ent) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= R) return;
    const Box b = box[r];
    int k = toff[r];
    for (int ty = b.y0 >> kTileShift; ty <= (b.y1 >> kTileShift); ty++)
        for (int tx = b.x0 >> kTileShift; tx <= (b.x1 >> kTileShift); tx++)
            ent[k++] = ((unsigned long long)(ty * tiles_x + tx) << 32) | (unsigned)r;
}

__global__ void k_tg_tile_bounds(int T, const unsigned long long* __restrict__ ent, int32_t* __restrict__ tstart,
                                 int32_t* __restrict__ tend) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= T) return;
    const int t = (int)(ent[i] >> 32);
    if (i == 0 || (int)(ent[i - 1] >> 32) != t) tstart[t] = i;
    if (i == T - 1 || (int)(ent[i + 1] >> 32) != t) tend[t] = i + 1;
}

__device__ __forceinline__ bool touch(const Box& a, const Box& b) {
    return !(a.x1 < b.x0 || b.x1 < a.x0 || a.y1 < b.y0 || b.y1 < a.y0);
}

// Visit every conflicting task of r exactly once: in the tile holding the lower-left corner of
// the intersection.  f(j) for each neighbour j; stops early when f returns false.
template <typename F>
__device__ __forceinline__ void for_neighbours(int r, const Box* box, const int32_t* tstart, const int32_t* tend,
                                               const unsigned long long* ent, int tiles_x, F f) {
    const Box b = box[r];
    for (int ty = b.y0 >> kTileShift; ty <= (b.y1 >> kTileShift); ty++)
        for (int tx = b.x0 >> kTileShift; tx <= (b.x1 >> kTileShift); tx++) {
            const int t = ty * tiles_x + tx;
            for (int k = tstart[t]; k < tend[t]; k++) {
                const int j = (int)(ent[k] & 0xFFFFFFFFull);
                if (j == r) continue;
                const Box c = box[j];
                if (!touch(b, c)) continue;
                const int cx = max(b.x0, c.x0), cy = max(b.y0, c.y0);
                if ((cx >> kTileShift) != tx || (cy >> kTileShift) != ty) continue;
                if (!f(j)) return;
            }
        }
}

// Root batch (one pass of Algorithm 1 = colour 0 of first-fit): rank-order dataflow, one
// thread per rank taken by ticket.  root[r]: 0 undecided, 1 root, 2 not root.
__global__ void k_tg_root(int R, const Box* __restrict__ box, const int32_t* __restrict__ tstart,
                          const int32_t* __restrict__ tend, const unsigned long long* __restrict__ ent, int tiles_x,
                          int* __restrict__ ticket, uint8_t* root) {
    for (;;) {
        const int r = atomicAdd(ticket, 1);
        if (r >= R) return;
        bool is_root = true;
        for_neighbours(r, box, tstart, tend, ent, tiles_x, [&](int j) {
            if (j > r) return true;
            int st;
            while ((st = *(volatile uint8_t*)&root[j]) == 0) __nanosleep(64);
            if (st == 1) { is_root = false; return false; }
            return true;
        });
        __threadfence();
        *(volatile uint8_t*)&root[r] = is_root ? 1 : 2;
    }
}

// successor counts (pass 0) and (source << 32 | target) edge keys (pass 1)
__global__ void k_tg_edges(int R, const Box* __restrict__ box, const int32_t* __restrict__ tstart,
                           const int32_t* __restrict__ tend, const unsigned long long* __restrict__ ent, int tiles_x,
                           const uint8_t* __restrict__ root, int32_t* __restrict__ cnt, const int32_t* __restrict__ eoff,
                           unsigned long long* __restrict__ ekeys, long long cap) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= R) return;
    const bool rr = root[r] == 1;
    int c = 0;
    const long long base = eoff ? eoff[r] : 0;
    for_neighbours(r, box, tstart, tend, ent, tiles_x, [&](int j) {
        const bool first = rr ? true : (root[j] == 1 ? false : r < j);
        if (first) {
            if (ekeys && base + c < cap) ekeys[base + c] = ((unsigned long long)r << 32) | (unsigned)j;
            c++;
        }
        return true;
    });
    if (!ekeys) cnt[r] = c;
}

__global__ void k_tg_root_u8(int R, const uint8_t* __restrict__ st, uint8_t* __restrict__ out) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r < R) out[r] = st[r] == 1 ? 1 : 0;
}

__global__ void k_tg_csr(long long E, const unsigned long long* __restrict__ ek, int32_t* __restrict__ succ) {
    const long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i < E) succ[i] = (int32_t)(ek[i] & 0xFFFFFFFFull);
}

}  // namespace

extern "C" FGR_API fgr_status fgr_overflow(fgr_grid* g, const fgr_nets* nets, const uint32_t* seg, const int32_t* zmid,
                                           uint8_t* violating, int32_t* rip_ids, int32_t* num_rip, int64_t* totals,
                                           void* stream) {
    if (!g || !nets || !num_rip || !totals) return fgr_set_error(FGR_ERR_INVALID, "NULL argument");
    if (g->broken) return fgr_set_error(FGR_ERR_STATE, "grid unusable after an earlier CUDA/NCCL error");
    const int N = nets->num_nets;
    if (N < 0) return fgr_set_error(FGR_ERR_INVALID, "negative sizes");
    if (N > 0 && (!seg || !violating || !rip_ids)) return fgr_set_error(FGR_ERR_INVALID, "NULL array");
    cudaStream_t st = (cudaStream_t)stream;
    FGR_CHECK_CUDA(g, cudaSetDevice(g->device));
    cudaError_t e;
    unsigned long long* tot = (unsigned long long*)fgr_scratch(g->s_rip[0], 64 + 4 * ((size_t)N + 1), &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "overflow scratch");
    int* nsel = (int*)(tot + 2);
    FGR_CHECK_CUDA(g, cudaMemsetAsync(tot, 0, 2 * sizeof(unsigned long long), st));
    const int blocks = g->num_sms * 8;
    k_ovf_totals<<<blocks, 256, 0, st>>>(g->view.h, tot);
    k_ovf_totals<<<blocks, 256, 0, st>>>(g->view.v, tot);
    FGR_CHECK_CUDA(g, cudaGetLastError());
    if (N > 0) {
        // a Z route needs its middle; without zmid the routes must be L shapes only
        if (!zmid && g->hyb_t1 <= g->hyb_t2) return fgr_set_error(FGR_ERR_INVALID, "hybrid patterns on: zmid required");
        k_ovf_nets<<<(unsigned)(((size_t)N * 32 + 255) / 256), 256, 0, st>>>(g->view, fgr_nets_view(nets), N, seg, zmid,
                                                                             violating);
        FGR_CHECK_CUDA(g, cudaGetLastError());
        size_t tb = 0;
        cub::CountingInputIterator<int32_t> ids(0);
        cub::DeviceSelect::Flagged(nullptr, tb, ids, violating, rip_ids, nsel, N, st);
        void* tmp = fgr_scratch(g->s_rip[1], tb, &e);
        if (e != cudaSuccess) return fgr_cuda_fail(g, e, "select scratch");
        FGR_CHECK_CUDA(g, cub::DeviceSelect::Flagged(tmp, tb, ids, violating, rip_ids, nsel, N, st));
    } else {
        FGR_CHECK_CUDA(g, cudaMemsetAsync(nsel, 0, sizeof(int), st));
    }
    unsigned long long h[2];
    int hn = 0;
    FGR_CHECK_CUDA(g, cudaMemcpyAsync(h, tot, sizeof(h), cudaMemcpyDeviceToHost, st));
    FGR_CHECK_CUDA(g, cudaMemcpyAsync(&hn, nsel, sizeof(int), cudaMemcpyDeviceToHost, st));
    FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));
    totals[0] = (int64_t)h[0];
    totals[1] = (int64_t)h[1];
    *num_rip = hn;
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_task_graph(fgr_grid* g, const fgr_nets* nets, const int32_t* tasks, int32_t count,
                                             int32_t* order, uint8_t* is_root, int32_t* succ_offset, int32_t* succ,
                                             int64_t capacity, int64_t* num_edges, void* stream) {
    if (!g || !nets || !num_edges) return fgr_set_error(FGR_ERR_INVALID, "NULL argument");
    if (g->broken) return fgr_set_error(FGR_ERR_STATE, "grid unusable after an earlier CUDA/NCCL error");
    if (count < 0 || capacity < 0) return fgr_set_error(FGR_ERR_INVALID, "negative sizes");
    if (!succ_offset || (count > 0 && (!tasks || !order || !is_root)) || (capacity > 0 && !succ))
        return fgr_set_error(FGR_ERR_INVALID, "NULL array");
    cudaStream_t st = (cudaStream_t)stream;
    FGR_CHECK_CUDA(g, cudaSetDevice(g->device));
    const int R = count;
    if (R == 0) {
        FGR_CHECK_CUDA(g, cudaMemsetAsync(succ_offset, 0, sizeof(int32_t), st));
        *num_edges = 0;
        return FGR_OK;
    }
    cudaError_t e;
    const NetsView nv = fgr_nets_view(nets);
    const int tiles_x = ((g->nx - 1) >> kTileShift) + 1, tiles_y = ((g->ny - 1) >> kTileShift) + 1;
    const int ntiles = tiles_x * tiles_y;
    // scratch: keys[2R] | box[R] | ntile[R+1] | toff[R+1] | tstart/tend[ntiles] | root[R] | ticket
    const size_t need = 16 * (size_t)R + sizeof(Box) * (size_t)R + 8 * ((size_t)R + 1) + 8 * (size_t)ntiles +
                        (size_t)R + 6 * 256;
    char* p = (char*)fgr_scratch(g->s_rip[2], need, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "task graph scratch");
    auto take = [&](size_t n) { char* q = p; p += (n + 255) & ~(size_t)255; return q; };
    unsigned long long* keys = (unsigned long long*)take(8 * (size_t)R);
    unsigned long long* keys_s = (unsigned long long*)take(8 * (size_t)R);
    Box* box = (Box*)take(sizeof(Box) * (size_t)R);
    int32_t* ntile = (int32_t*)take(4 * ((size_t)R + 1));
    int32_t* toff = (int32_t*)take(4 * ((size_t)R + 1));
    int32_t* tstart = (int32_t*)take(4 * (size_t)ntiles);
    int32_t* tend = (int32_t*)take(4 * (size_t)ntiles);
    uint8_t* rst = (uint8_t*)take((size_t)R + 4);
    int* ticket = (int*)take(4);
    const unsigned wb = (unsigned)(((size_t)R * 32 + 255) / 256), tbk = (unsigned)((R + 255) / 256);
    k_tg_keys<<<wb, 256, 0, st>>>(R, tasks, nv, keys);
    FGR_CHECK_CUDA(g, cudaGetLastError());
    size_t tb = 0, tb2 = 0;
    cub::DeviceRadixSort::SortKeys(nullptr, tb, keys, keys_s, R, 0, 64, st);
    cub::DeviceScan::ExclusiveSum(nullptr, tb2, ntile, toff, R + 1, st);
    void* tmp = fgr_scratch(g->s_rip[3], std::max(tb, tb2), &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "sort scratch");
    FGR_CHECK_CUDA(g, cub::DeviceRadixSort::SortKeys(tmp, tb, keys, keys_s, R, 0, 64, st));
    k_tg_boxes<<<wb, 256, 0, st>>>(R, keys_s, nv, order, box, ntile);
    FGR_CHECK_CUDA(g, cudaMemsetAsync(ntile + R, 0, sizeof(int32_t), st));
    FGR_CHECK_CUDA(g, cub::DeviceScan::ExclusiveSum(tmp, tb2, ntile, toff, R + 1, st));
    int T = 0;
    FGR_CHECK_CUDA(g, cudaMemcpyAsync(&T, toff + R, sizeof(int), cudaMemcpyDeviceToHost, st));
    FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));
    unsigned long long* ent = (unsigned long long*)fgr_scratch(g->s_rip[4], 16 * (size_t)T + 64, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "tile entries");
    unsigned long long* ent_s = ent + T;
    k_tg_tile_emit<<<tbk, 256, 0, st>>>(R, box, toff, tiles_x, ent);
    FGR_CHECK_CUDA(g, cudaGetLastError());
    int tbits = 1;
    while ((1LL << tbits) < ntiles) tbits++;
    cub::DeviceRadixSort::SortKeys(nullptr, tb, ent, ent_s, T, 0, 32 + tbits, st);
    tmp = fgr_scratch(g->s_rip[3], tb, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "sort scratch");
    FGR_CHECK_CUDA(g, cub::DeviceRadixSort::SortKeys(tmp, tb, ent, ent_s, T, 0, 32 + tbits, st));
    FGR_CHECK_CUDA(g, cudaMemsetAsync(tstart, 0, 4 * (size_t)ntiles, st));
    FGR_CHECK_CUDA(g, cudaMemsetAsync(tend, 0, 4 * (size_t)ntiles, st));
    k_tg_tile_bounds<<<(T + 255) / 256, 256, 0, st>>>(T, ent_s, tstart, tend);
    // root batch: persistent grid of resident threads taking ranks in order
    FGR_CHECK_CUDA(g, cudaMemsetAsync(rst, 0, (size_t)R, st));
    FGR_CHECK_CUDA(g, cudaMemsetAsync(ticket, 0, sizeof(int), st));
    k_tg_root<<<g->num_sms, 256, 0, st>>>(R, box, tstart, tend, ent_s, tiles_x, ticket, rst);
    k_tg_root_u8<<<tbk, 256, 0, st>>>(R, rst, is_root);
    // edges: counts, offsets, keys, sort, CSR
    k_tg_edges<<<tbk, 256, 0, st>>>(R, box, tstart, tend, ent_s, tiles_x, rst, ntile, nullptr, nullptr, 0);
    FGR_CHECK_CUDA(g, cudaMemsetAsync(ntile + R, 0, sizeof(int32_t), st));
    cub::DeviceScan::ExclusiveSum(nullptr, tb2, ntile, succ_offset, R + 1, st);
    tmp = fgr_scratch(g->s_rip[3], tb2, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "scan scratch");
    FGR_CHECK_CUDA(g, cub::DeviceScan::ExclusiveSum(tmp, tb2, ntile, succ_offset, R + 1, st));
    int hE = 0;
    FGR_CHECK_CUDA(g, cudaMemcpyAsync(&hE, succ_offset + R, sizeof(int), cudaMemcpyDeviceToHost, st));
    FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));
    *num_edges = hE;
    if (hE > capacity) return fgr_set_error(FGR_ERR_RANGE, "task graph has %d edges > capacity %lld", hE, (long long)capacity);
    if (hE > 0) {
        unsigned long long* ek = (unsigned long long*)fgr_scratch(g->s_rip[5], 16 * (size_t)hE + 64, &e);
        if (e != cudaSuccess) return fgr_cuda_fail(g, e, "edge keys");
        k_tg_edges<<<tbk, 256, 0, st>>>(R, box, tstart, tend, ent_s, tiles_x, rst, nullptr, succ_offset, ek, hE);
        int rbits = 1;
        while ((1LL << rbits) < R) rbits++;
        cub::DeviceRadixSort::SortKeys(nullptr, tb, ek, ek + hE, hE, 0, 32 + rbits, st);
        tmp = fgr_scratch(g->s_rip[3], tb, &e);
        if (e != cudaSuccess) return fgr_cuda_fail(g, e, "sort scratch");
        FGR_CHECK_CUDA(g, cub::DeviceRadixSort::SortKeys(tmp, tb, ek, ek + hE, hE, 0, 32 + rbits, st));
        k_tg_csr<<<(unsigned)((hE + 255) / 256), 256, 0, st>>>(hE, ek + hE, succ);
        FGR_CHECK_CUDA(g, cudaGetLastError());
    }
    FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));
    return FGR_OK;
}
