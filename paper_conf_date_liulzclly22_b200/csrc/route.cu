// route.cu — the pattern-routing stage driver: batches in sequence (PAPER.md
// L504-512, Fig. 7 "kernels invoked sequentially, each processing one batch"),
// each batch = [cost refresh of the segments the previous batch dirtied] ->
// [tree DP + backtrack + commit].  Multi-GPU (not in the paper; north_star): the
// grid is replicated, each batch's nets are split across ranks, the per-node
// route records of the batch are exchanged with one NCCL all-reduce (records of
// other ranks' nets are zero), and every rank commits every net of the batch, so
// all replicas stay bitwise identical to the 1-GPU result (nets of one batch are
// independent: reading R13).
#include <cub/cub.cuh>

#include <cstdlib>
#include <cstdint>
#include <cstring>

#include "fgr_internal.cuh"

namespace {

// route_batch: split a net list into large (> 32 nodes) | midL (9..32) | midS (3..8) | two (2 nodes)
__device__ __forceinline__ int size_class(int m) {
    return m > FGR_SMALL_NET ? 0 : (m > FGR_MID_NET ? 1 : (m > 2 ? 2 : 3));   // m <= 2 (incl. trivial) -> 3
}

__global__ void k_classify(int count, const int32_t* __restrict__ ids, const int32_t* __restrict__ off,
                           int32_t* __restrict__ tmp, int* __restrict__ ctr /* [0..3] class counts, [4] maxm */) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= count) return;
    const int id = ids[i];
    const int m = off[id + 1] - off[id];
    const int k = size_class(m);
    tmp[(size_t)k * count + atomicAdd(&ctr[k], 1)] = id;
    if (k == 0) atomicMax(&ctr[4], m);
}

__global__ void k_concat4(int count, const int32_t* __restrict__ tmp, const int* __restrict__ ctr,
                          int32_t* __restrict__ out) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= count) return;
    int k = 0, base = 0;
    while (k < 3 && i >= base + ctr[k]) { base += ctr[k]; k++; }
    out[i] = tmp[(size_t)k * count + (i - base)];
}

__global__ void k_net_sizes(int n, const int32_t* __restrict__ order, const int32_t* __restrict__ off,
                            int32_t* __restrict__ sizes) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) sizes[i] = off[order[i] + 1] - off[order[i]];
}

__global__ void k_batch_info(int B, const int32_t* __restrict__ boff, const int32_t* __restrict__ order,
                             const int32_t* __restrict__ off, const int16_t* __restrict__ x,
                             const int16_t* __restrict__ y, const int32_t* __restrict__ par,
                             int* __restrict__ nlarge, int* __restrict__ maxm, unsigned long long* __restrict__ segb,
                             int* __restrict__ ntwo, int* __restrict__ n9, unsigned long long* __restrict__ keys,
                             int* __restrict__ lsplit, int lim) {
    // one block per batch
    const int b = blockIdx.x;
    if (b >= B) return;
    int nl = 0, mm = 0, n2 = 0, nn9 = 0, ls[5] = {0, 0, 0, 0, 0};
    unsigned long long sb = 0;
    for (int i = boff[b] + threadIdx.x; i < boff[b + 1]; i += blockDim.x) {
        const int id = order[i];
        const int a0 = off[id], m = off[id + 1] - a0;
        if (m > FGR_SMALL_NET) { nl++; mm = max(mm, m); }
        ls[0] += m > lim; ls[1] += m > 512; ls[2] += m > 256; ls[3] += m > 128; ls[4] += m > 64;
        if (m <= 2) n2++;   // the 2-node kernel also finishes trivial nets
        if (m > FGR_MID_NET && m <= FGR_SMALL_NET) nn9++;
        for (int j = 1; j < m; j++) {
            const int u = a0 + par[a0 + j];
            sb += (unsigned)((abs(x[a0 + j] - x[u]) >> 5) + (abs(y[a0 + j] - y[u]) >> 5) + 4);
        }
        // exec order inside the batch: larger nets first (same key layout as fgr_plan)
        const unsigned inv = 2047u - (unsigned)min(m, 2047);
        keys[i] = ((unsigned long long)b << 42) | ((unsigned long long)inv << 31) | (unsigned)id;
    }
    atomicAdd(&nlarge[b], nl);
    atomicMax(&maxm[b], mm);
    atomicAdd(&segb[b], sb);
    atomicAdd(&ntwo[b], n2);
    atomicAdd(&n9[b], nn9);
    for (int k = 0; k < 5; k++) atomicAdd(&lsplit[5 * b + k], ls[k]);
}

__global__ void k_large_list(int n, const int32_t* __restrict__ exec, const int32_t* __restrict__ off,
                             int32_t* __restrict__ out, int* __restrict__ cnt, int minm) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const int id = exec[i];
    const int m = off[id + 1] - off[id];
    if (m > FGR_SMALL_NET && m <= minm) out[atomicAdd(cnt, 1)] = id;   // the heavy-path / dataflow kernels' nets
    if (m > minm) out[n + atomicAdd(cnt + 1, 1)] = id;                 // the nets that take k_dp_hld
}

__global__ void k_keys_to_ids(int n, const unsigned long long* __restrict__ keys, int32_t* __restrict__ ids) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) ids[i] = (int32_t)(keys[i] & 0x7FFFFFFFu);
}

__global__ void k_scatter_records(int n, const int32_t* __restrict__ order, const int32_t* __restrict__ off,
                                  const int32_t* __restrict__ rec_off, const uint32_t* __restrict__ rec_seg,
                                  const uint32_t* __restrict__ rec_cost, uint32_t* __restrict__ seg_out,
                                  uint32_t* __restrict__ cost_out) {
    const int warp = (int)((blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5);
    if (warp >= n) return;
    const int id = order[warp];
    const int a0 = off[id], m = off[id + 1] - a0;
    for (int j = lane_id(); j < m; j += 32) seg_out[a0 + j] = rec_seg[rec_off[warp] + j];
    if (lane_id() == 0) cost_out[id] = rec_cost[warp];
}

inline size_t a16h(size_t b) { return (b + 15) & ~(size_t)15; }

bool nets_equal(const fgr_nets& a, const fgr_nets& b) {
    return a.num_nets == b.num_nets && a.num_nodes == b.num_nodes && a.node_offset == b.node_offset && a.x == b.x &&
           a.y == b.y && a.pin_lo == b.pin_lo && a.pin_hi == b.pin_hi && a.parent == b.parent;
}

}  // namespace

// Refresh before a DP launch: a full rescan after set_demand/creation, else only
// the segments the last commit dirtied (bounded by `max_tasks`).
static cudaError_t refresh_before_dp(fgr_grid* g, cudaStream_t st, long long max_tasks) {
    if (g->full_dirty) {
        g->full_dirty = false;
        return fgr_launch_refresh_sized(g, st, true, 0);
    }
    return fgr_launch_refresh_sized(g, st, false, max_tasks);
}

// first index i in [lo, hi] with pre[i] - pre[lo] >= target (pre non-decreasing)
static int32_t split_point(const int64_t* pre, int32_t lo, int32_t hi, int64_t target) {
    int32_t a = lo, b = hi;
    while (a < b) {
        const int32_t mid = a + (b - a) / 2;
        if (pre[mid] - pre[lo] >= target) b = mid; else a = mid + 1;
    }
    return a;
}

extern "C" FGR_API fgr_status fgr_split_batch(int32_t count, int32_t nlarge, const int64_t* edge_prefix, int32_t split_min,
                                              int32_t rank, int32_t world, int32_t* out) {
    if (!out || count < 0 || nlarge < 0 || nlarge > count || world < 1 || rank < 0 || rank >= world)
        return fgr_set_error(FGR_ERR_INVALID, "bad split arguments");
    if (count < split_min) {   // too small to pay an exchange: every rank routes the whole batch
        out[0] = 0; out[1] = nlarge; out[2] = nlarge; out[3] = count; out[4] = 1;
        return FGR_OK;
    }
    out[4] = 0;
    if (!edge_prefix) {
        const long long ns = count - nlarge;
        out[0] = (int32_t)((long long)nlarge * rank / world);
        out[1] = (int32_t)((long long)nlarge * (rank + 1) / world);
        out[2] = nlarge + (int32_t)(ns * rank / world);
        out[3] = nlarge + (int32_t)(ns * (rank + 1) / world);
        return FGR_OK;
    }
    // balanced by tree edges: contiguous chunks of the large and of the small nets
    const int64_t el = edge_prefix[nlarge] - edge_prefix[0], es = edge_prefix[count] - edge_prefix[nlarge];
    out[0] = rank == 0 ? 0 : split_point(edge_prefix, 0, nlarge, (el * rank + world - 1) / world);
    out[1] = rank == world - 1 ? nlarge : split_point(edge_prefix, 0, nlarge, (el * (rank + 1) + world - 1) / world);
    out[2] = rank == 0 ? nlarge : split_point(edge_prefix, nlarge, count, (es * rank + world - 1) / world);
    out[3] = rank == world - 1 ? count : split_point(edge_prefix, nlarge, count, (es * (rank + 1) + world - 1) / world);
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_set_exchange(fgr_grid* g, int32_t split_min, int32_t emulate_world) {
    if (!g) return fgr_set_error(FGR_ERR_INVALID, "grid is NULL");
    if (split_min < 0 || emulate_world < 0 || emulate_world > 1024)
        return fgr_set_error(FGR_ERR_INVALID, "bad exchange settings %d / %d", split_min, emulate_world);
    g->split_min = split_min;
    g->emu_world = emulate_world;
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_set_graph(fgr_grid* g, int32_t on) {
    if (!g) return fgr_set_error(FGR_ERR_INVALID, "grid is NULL");
    g->rg.use = on != 0;
    if (!g->rg.use && g->rg.exec) { cudaGraphExecDestroy(g->rg.exec); g->rg.exec = nullptr; }
    g->rg.key.clear();
    g->rg.seen_key.clear();
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_set_dp_policy(fgr_grid* g, int32_t policy, int32_t flow_max) {
    if (!g) return fgr_set_error(FGR_ERR_INVALID, "grid is NULL");
    if (policy != FGR_DP_AUTO && policy != FGR_DP_HEAVY && policy != FGR_DP_HLD)
        return fgr_set_error(FGR_ERR_INVALID, "unknown DP policy %d", policy);
    if (flow_max < FGR_SMALL_NET + 1 || flow_max > 65535) return fgr_set_error(FGR_ERR_INVALID, "flow_max %d out of range", flow_max);
    if (policy != g->dp_policy) {   // the decompositions and the size buckets depend on the policy
        g->cache.prep_valid = false;
        g->cache.valid = false;
    }
    g->dp_policy = policy;
    g->flow_max = flow_max;
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_set_pattern(fgr_grid* g, int32_t hybrid_t1, int32_t hybrid_t2) {
    if (!g) return fgr_set_error(FGR_ERR_INVALID, "grid is NULL");
    if (hybrid_t1 <= hybrid_t2 && (hybrid_t1 < 0 || hybrid_t2 > 2 * 32767))
        return fgr_set_error(FGR_ERR_INVALID, "hybrid window [%d, %d] out of range", hybrid_t1, hybrid_t2);
    g->hyb_t1 = hybrid_t1;
    g->hyb_t2 = hybrid_t2;
    g->hy.cached = false;
    return FGR_OK;
}

static fgr_status hld_prep_list(fgr_grid* g, const fgr_nets* nets, const int32_t* list, int nl, int maxm, cudaStream_t st,
                                HldPrep* out);

extern "C" FGR_API fgr_status fgr_route_batch(fgr_grid* g, const fgr_nets* nets, const int32_t* net_ids, int32_t count,
                                              uint32_t* seg_out, uint32_t* net_cost, void* stream) {
    return fgr_route_batch_ex(g, nets, net_ids, count, seg_out, nullptr, net_cost, stream);
}

extern "C" FGR_API fgr_status fgr_route_batch_ex(fgr_grid* g, const fgr_nets* nets, const int32_t* net_ids, int32_t count,
                                                 uint32_t* seg_out, int32_t* zmid_out, uint32_t* net_cost, void* stream) {
    if (!g || !nets) return fgr_set_error(FGR_ERR_INVALID, "NULL argument");
    if (g->broken) return fgr_set_error(FGR_ERR_STATE, "grid unusable after an earlier CUDA/NCCL error");
    if (count < 0) return fgr_set_error(FGR_ERR_INVALID, "count < 0");
    if (count == 0) return FGR_OK;
    if (!net_ids || !seg_out || !net_cost) return fgr_set_error(FGR_ERR_INVALID, "NULL array");
    cudaStream_t st = (cudaStream_t)stream;
    FGR_CHECK_CUDA(g, cudaSetDevice(g->device));
    cudaError_t e;
    int32_t* list = (int32_t*)fgr_scratch(g->s_rec[0], sizeof(int32_t) * (size_t)count * 5 + 64, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "route_batch scratch");
    int32_t* tmp = list + count;
    int* ctr = (int*)(list + 5 * (size_t)count);
    FGR_CHECK_CUDA(g, cudaMemsetAsync(ctr, 0, 8 * sizeof(int), st));
    k_classify<<<(count + 255) / 256, 256, 0, st>>>(count, net_ids, nets->node_offset, tmp, ctr);
    k_concat4<<<(count + 255) / 256, 256, 0, st>>>(count, tmp, ctr, list);
    FGR_CHECK_CUDA(g, cudaGetLastError());
    int hc[8];
    FGR_CHECK_CUDA(g, cudaMemcpyAsync(hc, ctr, sizeof(hc), cudaMemcpyDeviceToHost, st));
    FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));
    const NetsView nv = fgr_nets_view(nets);
    g->hy.cached = false;   // the hybrid tables below cover this batch only
    fgr_status s = fgr_hyb_prepare(g, st, nv, nets->num_nets, nets->num_nodes, list, count, nullptr, 1, zmid_out);
    if (s != FGR_OK) return s;
    Prep bp{};
    if (hc[0] > 0 && (hc[4] > fgr_top_limit(g) || g->dp_policy != FGR_DP_HEAVY)) {
        g->cache.prep_valid = false;   // s_hldp now holds this batch's decomposition
        s = hld_prep_list(g, nets, list, hc[0], hc[4], st, &bp.hld);
        if (s != FGR_OK) return s;
    }
    FGR_CHECK_CUDA(g, refresh_before_dp(g, st, g->total_segs));
    FGR_CHECK_CUDA(g, fgr_launch_hyb_tm(g, st, nv, 0, g->hy.nslots));
    FGR_CHECK_CUDA(g, fgr_launch_dp(g, st, nv, list, hc[0], hc[1], hc[2], hc[3], hc[4], seg_out, net_cost, nullptr,
                                    nullptr, nullptr, 0, true, &bp));
    FGR_CHECK_CUDA(g, fgr_launch_hyb_zmid(g, st, seg_out, zmid_out));
    return FGR_OK;
}

// Host mirrors of per-batch launch sizes: from fgr_plan's cache, or rebuilt (one sync).
static fgr_status batch_info(fgr_grid* g, const fgr_nets* nets, const int32_t* order, const int32_t* batch_offset,
                             int B, cudaStream_t st) {
    PlanCache& c = g->cache;
    if (c.valid && c.num_batches == B && c.order == order && c.batch_offset == batch_offset &&
        nets_equal(c.nets, *nets))
        return FGR_OK;
    cudaError_t e;
    const int R = 0;   // net count of the batches is read back below
    (void)R;
    void* p = fgr_scratch(g->s_rec[1], (size_t)B * 44 + 64, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "batch info scratch");
    unsigned long long* d_segb = (unsigned long long*)p;
    int* d_nl = (int*)(d_segb + B);
    int* d_mm = d_nl + B;
    int* d_n2 = d_mm + B;
    int* d_n9 = d_n2 + B;
    int* d_ls = d_n9 + B;
    FGR_CHECK_CUDA(g, cudaMemsetAsync(p, 0, (size_t)B * 44, st));
    FGR_CHECK_CUDA(g, fgr_mirrors_reserve(c, B));
    FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_off, batch_offset, sizeof(int) * (B + 1), cudaMemcpyDeviceToHost, st));
    FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));
    const int nb = B > 0 ? c.h_off[B] : 0;
    // the exec order is re-sorted inside each batch (larger nets first): any order the caller gives is fine
    unsigned long long* keys = (unsigned long long*)fgr_scratch(g->s_plan[0], 16 * ((size_t)nb + 1), &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "exec keys");
    unsigned long long* keys_s = keys + nb;
    int32_t* exec = (int32_t*)fgr_scratch(g->s_plan[13], 4 * ((size_t)nb + 1), &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "exec order");
    if (B > 0) {
        k_batch_info<<<B, 256, 0, st>>>(B, batch_offset, order, nets->node_offset, nets->x, nets->y, nets->parent,
                                        d_nl, d_mm, d_segb, d_n2, d_n9, keys, d_ls, fgr_top_limit(g));
        FGR_CHECK_CUDA(g, cudaGetLastError());
        int bits = 42;
        while ((1LL << (bits - 42)) <= B) bits++;
        size_t tb = 0;
        cub::DeviceRadixSort::SortKeys(nullptr, tb, keys, keys_s, nb, 0, bits, st);
        void* tmp = fgr_scratch(g->s_plan[8], tb, &e);
        if (e != cudaSuccess) return fgr_cuda_fail(g, e, "exec sort scratch");
        FGR_CHECK_CUDA(g, cub::DeviceRadixSort::SortKeys(tmp, tb, keys, keys_s, nb, 0, bits, st));
        k_keys_to_ids<<<(nb + 255) / 256, 256, 0, st>>>(nb, keys_s, exec);
        FGR_CHECK_CUDA(g, cudaGetLastError());
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_nlarge, d_nl, sizeof(int) * B, cudaMemcpyDeviceToHost, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_maxm, d_mm, sizeof(int) * B, cudaMemcpyDeviceToHost, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_segb, d_segb, sizeof(long long) * B, cudaMemcpyDeviceToHost, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_ntwo, d_n2, sizeof(int) * B, cudaMemcpyDeviceToHost, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_n9, d_n9, sizeof(int) * B, cudaMemcpyDeviceToHost, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(c.h_lsplit, d_ls, sizeof(int) * 5 * B, cudaMemcpyDeviceToHost, st));
    }
    FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));
    c.valid = true;
    c.prep_valid = false;
    g->hy.cached = false;
    c.exec = exec;
    c.nets = *nets;
    c.order = order;
    c.batch_offset = batch_offset;
    c.num_batches = B;
    return FGR_OK;
}

// Large-net tree analysis once per stage (k_large_prep), reused by every batch's k_dp_large.
// Heavy-path decomposition of a list of large nets (k_hld_prep) into g->s_hldp.
static fgr_status hld_prep_list(fgr_grid* g, const fgr_nets* nets, const int32_t* list, int nl, int maxm, cudaStream_t st,
                                HldPrep* out) {
    const size_t M = (size_t)nets->num_nodes, N = (size_t)nets->num_nets;
    cudaError_t e;
    char* p = (char*)fgr_scratch(g->s_hldp, 6 * a16h(2 * M) + 2 * a16h(M) + a16h(4 * N) + 64, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "hld prep arrays");
    auto take = [&](size_t b) { char* q = p; p += a16h(b); return q; };
    uint16_t* hv = (uint16_t*)take(2 * M); uint16_t* cs = (uint16_t*)take(2 * M); uint16_t* cl = (uint16_t*)take(2 * M);
    uint16_t* pn = (uint16_t*)take(2 * M); uint16_t* po = (uint16_t*)take(2 * M);
    uint8_t* pr = (uint8_t*)take(M);
    int32_t* info = (int32_t*)take(4 * N);
    uint8_t* ld = (uint8_t*)take(M);
    uint16_t* lf = (uint16_t*)take(2 * M);
    FGR_CHECK_CUDA(g, fgr_launch_hld_prep(g, st, fgr_nets_view(nets), list, nl, maxm, hv, cs, cl, pn, po, pr, info, ld, lf));
    *out = HldPrep{hv, cs, cl, pn, po, pr, info, ld, lf};
    return FGR_OK;
}

// Large-net tree analyses once per stage, reused by every batch's large-net DP launches: the
// heavy-path tables of k_dp_flow / k_dp_large (k_large_prep) for the nets they route, and the
// decomposition of k_dp_hld (k_hld_prep) for the nets it routes (fgr_set_dp_policy).
static fgr_status ensure_prep(fgr_grid* g, const fgr_nets* nets, int B, cudaStream_t st) {
    PlanCache& c = g->cache;
    if (c.prep_valid) return FGR_OK;
    const int R = B > 0 ? c.h_off[B] : 0;
    const int lim = fgr_top_limit(g);
    int maxm = 0, nl = 0, nh = 0;
    for (int b = 0; b < B; b++) {
        maxm = c.h_maxm[b] > maxm ? c.h_maxm[b] : maxm;
        nl += c.h_nlarge[b];
        nh += c.h_lsplit[5 * b];
    }
    const bool all_hld = g->dp_policy != FGR_DP_HEAVY;   // k_dp_tree and k_dp_hld both read the HLD decomposition
    if (all_hld) nh = nl;
    c.prep = Prep{};
    if (nl == 0) { c.prep_valid = true; return FGR_OK; }
    const size_t M = (size_t)nets->num_nodes, N = (size_t)nets->num_nets;
    cudaError_t e;
    char* p = (char*)fgr_scratch(g->s_prep, 6 * 2 * M + 4 * N + 8 * (size_t)R + 64 + 6 * 16, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "prep arrays");
    auto take16 = [&](size_t n) { uint16_t* q = (uint16_t*)p; p += (2 * n + 15) & ~(size_t)15; return q; };
    uint16_t* cs = take16(M); uint16_t* cl = take16(M); uint16_t* hv = take16(M); uint16_t* bot = take16(M);
    uint16_t* pq = take16(M);
    uint16_t* rpos = take16(M);
    int32_t* np = (int32_t*)p; p += (4 * N + 15) & ~(size_t)15;
    int32_t* list = (int32_t*)p; p += 8 * (size_t)R;   // [R] nets of k_large_prep | [R] nets of k_hld_prep
    int* cnt = (int*)p;
    FGR_CHECK_CUDA(g, cudaMemsetAsync(cnt, 0, 2 * sizeof(int), st));
    k_large_list<<<(R + 255) / 256, 256, 0, st>>>(R, c.exec, nets->node_offset, list, cnt, all_hld ? FGR_SMALL_NET : lim);
    FGR_CHECK_CUDA(g, cudaGetLastError());
    if (!all_hld && nl > nh) {
        FGR_CHECK_CUDA(g, fgr_launch_large_prep(g, st, fgr_nets_view(nets), list, nl - nh, min(maxm, lim), cs, cl, hv, bot,
                                                pq, rpos, np));
        c.prep = Prep{cs, cl, hv, bot, pq, np, rpos, HldPrep{}};
    }
    if (nh > 0) {
        fgr_status s = hld_prep_list(g, nets, list + R, nh, maxm, st, &c.prep.hld);
        if (s != FGR_OK) return s;
    }
    c.prep_valid = true;
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_route_all(fgr_grid* g, const fgr_nets* nets, const int32_t* order,
                                            const int32_t* batch_offset, int32_t num_batches, uint32_t* seg_out,
                                            uint32_t* net_cost, void* stream) {
    return fgr_route_all_ex(g, nets, order, batch_offset, num_batches, seg_out, nullptr, net_cost, stream);
}

// Hybrid tables for the stage (cached with the plan: same nets, exec order and window).
static fgr_status ensure_hyb(fgr_grid* g, const fgr_nets* nets, const int32_t* batch_offset, int B, cudaStream_t st) {
    HybState& h = g->hy;
    const PlanCache& c = g->cache;
    if (h.cached && h.key_exec == c.exec && h.key_t1 == g->hyb_t1 && h.key_t2 == g->hyb_t2) return FGR_OK;
    const int R = B > 0 ? c.h_off[B] : 0;
    fgr_status s = fgr_hyb_prepare(g, st, fgr_nets_view(nets), nets->num_nets, nets->num_nodes, c.exec, R, batch_offset,
                                   B, nullptr);
    if (s != FGR_OK) return s;
    h.cached = true;
    h.key_exec = c.exec;
    h.key_t1 = g->hyb_t1;
    h.key_t2 = g->hyb_t2;
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_route_all_ex(fgr_grid* g, const fgr_nets* nets, const int32_t* order,
                                               const int32_t* batch_offset, int32_t num_batches, uint32_t* seg_out,
                                               int32_t* zmid_out, uint32_t* net_cost, void* stream) {
    if (!g || !nets) return fgr_set_error(FGR_ERR_INVALID, "NULL argument");
    if (g->broken) return fgr_set_error(FGR_ERR_STATE, "grid unusable after an earlier CUDA/NCCL error");
    const int B = num_batches, N = nets->num_nets, M = nets->num_nodes;
    if (B < 0 || N < 0 || M < 0) return fgr_set_error(FGR_ERR_INVALID, "negative sizes");
    if (N > 0 && (!order || !batch_offset || !seg_out || !net_cost))
        return fgr_set_error(FGR_ERR_INVALID, "NULL array");
    cudaStream_t st = (cudaStream_t)stream;
    FGR_CHECK_CUDA(g, cudaSetDevice(g->device));
    fgr_status s = batch_info(g, nets, order, batch_offset, B, st);
    if (s != FGR_OK) return s;
    s = ensure_prep(g, nets, B, st);
    if (s != FGR_OK) return s;
    s = ensure_hyb(g, nets, batch_offset, B, st);
    if (s != FGR_OK) return s;
    const PlanCache& c = g->cache;
    const HybState& hy = g->hy;
    if (M > 0) FGR_CHECK_CUDA(g, cudaMemsetAsync(seg_out, 0xFF, sizeof(uint32_t) * (size_t)M, st));
    if (M > 0 && zmid_out) FGR_CHECK_CUDA(g, cudaMemsetAsync(zmid_out, 0xFF, sizeof(int32_t) * (size_t)M, st));
    if (N > 0) FGR_CHECK_CUDA(g, cudaMemsetAsync(net_cost, 0, sizeof(uint32_t) * (size_t)N, st));
    const NetsView nv = fgr_nets_view(nets);
    g->stats.num_batches = B;
    g->stats.world = g->world;
    g->stats.rank = g->rank;
    g->stats.dp_nets = B > 0 ? c.h_off[B] : 0;
    g->stats.dp_edges = (int64_t)M - N;   // every net is a tree: sum of (nodes - 1)
    g->stats.exchanged_batches = 0;
    g->stats.kernel_launches = 0;
    FGR_CHECK_CUDA(g, cudaMemsetAsync(g->d_stats, 0, 4 * sizeof(unsigned long long), st));
    const bool emu = !g->comm && g->emu_world > 1;
    if (!g->comm && !emu) {
        // the batch loop (batches in sequence), replayed as a CUDA Graph when
        // nothing its launches depend on changed since the previous call (fgr_set_graph)
        auto loop = [&](cudaStream_t st) -> cudaError_t {
            cudaError_t e2;
            for (int b = 0; b < B; b++) {
                const long long bound = b > 0 ? c.h_segb[b - 1] : (long long)g->total_segs;
                if ((e2 = refresh_before_dp(g, st, bound)) != cudaSuccess) return e2;
                if (hy.active && (e2 = fgr_launch_hyb_tm(g, st, nv, hy.boff[b], hy.boff[b + 1] - hy.boff[b])) != cudaSuccess)
                    return e2;
                const int o0 = c.h_off[b], cnt = c.h_off[b + 1] - o0, nl = c.h_nlarge[b], n2 = c.h_ntwo[b], n9 = c.h_n9[b];
                if ((e2 = fgr_launch_dp(g, st, nv, c.exec + o0, nl, n9, cnt - nl - n9 - n2, n2, c.h_maxm[b], seg_out,
                                        net_cost, nullptr, nullptr, nullptr, 0, true, &c.prep, c.h_lsplit + 5 * b)) !=
                    cudaSuccess)
                    return e2;
            }
            return fgr_launch_hyb_zmid(g, st, seg_out, zmid_out);
        };
        RouteGraph& rg = g->rg;
        g->stats.graph_mode = 0;
        if (!rg.use || g->prof.on || B == 0) {
            FGR_CHECK_CUDA(g, loop(st));
            return FGR_OK;
        }
        std::vector<long long> key = {(long long)(uintptr_t)c.exec, B, (long long)(uintptr_t)nets->node_offset,
                                      (long long)(uintptr_t)nets->x, (long long)(uintptr_t)nets->y,
                                      (long long)(uintptr_t)nets->pin_lo, (long long)(uintptr_t)nets->pin_hi,
                                      (long long)(uintptr_t)nets->parent, N, M, (long long)(uintptr_t)seg_out,
                                      (long long)(uintptr_t)zmid_out, (long long)(uintptr_t)net_cost,
                                      (long long)(uintptr_t)st, g->dp_policy, g->flow_max, hy.active ? 1 : 0,
                                      g->hyb_t1, g->hyb_t2, g->full_dirty ? 1 : 0, (long long)g_scratch_gen};
        std::vector<long long> mir;
        mir.reserve((size_t)B * 12 + 1);
        for (int b = 0; b <= B; b++) mir.push_back(c.h_off[b]);
        for (int b = 0; b < B; b++) {
            mir.push_back(c.h_nlarge[b]); mir.push_back(c.h_maxm[b]); mir.push_back(c.h_ntwo[b]);
            mir.push_back(c.h_n9[b]); mir.push_back(c.h_segb[b]);
            for (int k = 0; k < 5; k++) mir.push_back(c.h_lsplit[5 * b + k]);
        }
        if (hy.active)
            for (int x : hy.boff) mir.push_back(x);
        if (rg.exec && key == rg.key && mir == rg.mirror) {
            FGR_CHECK_CUDA(g, cudaGraphLaunch(rg.exec, st));
            g->full_dirty = false;
            g->stats.kernel_launches += rg.launches;
            g->stats.graph_mode = 2;
            return FGR_OK;
        }
        if (key == rg.seen_key && mir == rg.seen_mirror) {
            // second call with these inputs (every scratch buffer is sized): capture the loop on the
            // grid's private stream (the caller's may be the legacy stream, which cannot be captured),
            // then launch the graph on the caller's stream
            if (rg.exec) { cudaGraphExecDestroy(rg.exec); rg.exec = nullptr; }
            const bool fd = g->full_dirty;
            const long long l0 = g->stats.kernel_launches;
            cudaGraph_t graph = nullptr;
            cudaError_t e2 = cudaSuccess;
            if (!rg.cap) e2 = cudaStreamCreateWithFlags(&rg.cap, cudaStreamNonBlocking);
            if (e2 == cudaSuccess) e2 = cudaStreamBeginCapture(rg.cap, cudaStreamCaptureModeThreadLocal);
            if (e2 == cudaSuccess) {
                const cudaError_t el = loop(rg.cap);
                e2 = cudaStreamEndCapture(rg.cap, &graph);
                if (el != cudaSuccess) e2 = el;
            }
            if (e2 == cudaSuccess && g_scratch_gen == (unsigned long long)key[key.size() - 1])
                e2 = cudaGraphInstantiate(&rg.exec, graph, 0);
            else if (e2 == cudaSuccess)
                e2 = cudaErrorStreamCaptureInvalidated;   // a buffer moved during capture: not reusable
            if (graph) cudaGraphDestroy(graph);
            if (e2 == cudaSuccess) {
                rg.key = key;
                rg.mirror = mir;
                rg.launches = g->stats.kernel_launches - l0;
                FGR_CHECK_CUDA(g, cudaGraphLaunch(rg.exec, st));
                g->stats.graph_mode = 1;
                return FGR_OK;
            }
            // capture failed: clear the sticky error state of this attempt and run the loop directly
            // (the reason stays readable through fgr_last_error; the call itself succeeds)
            if (rg.exec) { cudaGraphExecDestroy(rg.exec); rg.exec = nullptr; }
            (void)cudaGetLastError();
            fgr_set_error(FGR_OK, "batch-loop graph capture failed (%s); direct launches from now on",
                          cudaGetErrorString(e2));
            g->full_dirty = fd;
            g->stats.kernel_launches = l0;
            rg.use = false;
        }
        FGR_CHECK_CUDA(g, loop(st));
        key.back() = (long long)g_scratch_gen;   // buffers the direct run sized are in place for the next call
        rg.seen_key = key;
        rg.seen_mirror = mir;
        return FGR_OK;
    }
    // ---- multi-GPU: split each batch by tree edges, exchange route records, commit everywhere.
    // Batches with fewer than split_min nets are routed whole on every rank (no exchange: the
    // routes are deterministic).  emu: all `world` ranks' chunks run on this device into the
    // shared records, which then hold what the NCCL SUM would (test mode, fgr_set_exchange).
    const int W = emu ? g->emu_world : g->world;
    cudaError_t e;
    const int R = B > 0 ? c.h_off[B] : 0;
    int32_t* rec_off = (int32_t*)fgr_scratch(g->s_rec[2], sizeof(int32_t) * ((size_t)R + 1) * 2 + 64, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "record offsets");
    int32_t* sizes = rec_off + R + 1;
    if (R > 0) {
        k_net_sizes<<<(R + 255) / 256, 256, 0, st>>>(R, c.exec, nets->node_offset, sizes);
        FGR_CHECK_CUDA(g, cudaGetLastError());
    }
    FGR_CHECK_CUDA(g, cudaMemsetAsync(sizes + R, 0, sizeof(int32_t), st));
    std::vector<int32_t> h_sz((size_t)R + 1);
    if (R > 0) FGR_CHECK_CUDA(g, cudaMemcpyAsync(h_sz.data(), sizes, sizeof(int32_t) * (size_t)R, cudaMemcpyDeviceToHost, st));
    size_t tb = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, tb, sizes, rec_off, R + 1, st);
    void* tmp = fgr_scratch(g->s_plan[8], tb, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "scan scratch");
    FGR_CHECK_CUDA(g, cub::DeviceScan::ExclusiveSum(tmp, tb, sizes, rec_off, R + 1, st));
    std::vector<int> h_roff((size_t)B + 1);
    for (int b = 0; b <= B; b++)
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(h_roff.data() + b, rec_off + c.h_off[b], sizeof(int), cudaMemcpyDeviceToHost, st));
    FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));
    std::vector<int64_t> h_epre((size_t)R + 1);   // tree-edge prefix over the exec order
    h_epre[0] = 0;
    for (int i = 0; i < R; i++) h_epre[(size_t)i + 1] = h_epre[i] + (h_sz[i] - 1);
    const size_t nrec = (size_t)h_roff[B];
    uint32_t* rec = (uint32_t*)fgr_scratch(g->s_rec[3], sizeof(uint32_t) * (nrec + (size_t)R + 1), &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "records");
    uint32_t* rec_cost = rec + nrec;
    FGR_CHECK_CUDA(g, cudaMemsetAsync(rec, 0, sizeof(uint32_t) * (nrec + (size_t)R + 1), st));
    g->stats.exchanged_batches = 0;
    for (int b = 0; b < B; b++) {
        const long long bound = b > 0 ? c.h_segb[b - 1] : (long long)g->total_segs;
        FGR_CHECK_CUDA(g, refresh_before_dp(g, st, bound));
        // every rank builds the batch's hybrid matrices: the commit of remote routes reads their Z argmins
        if (hy.active) FGR_CHECK_CUDA(g, fgr_launch_hyb_tm(g, st, nv, hy.boff[b], hy.boff[b + 1] - hy.boff[b]));
        const int o0 = c.h_off[b], cnt = c.h_off[b + 1] - o0, nl = c.h_nlarge[b], n2 = c.h_ntwo[b], n9 = c.h_n9[b];
        int32_t sp[5];
        fgr_split_batch(cnt, nl, h_epre.data() + o0, g->split_min, 0, W, sp);
        if (sp[4]) {   // routed whole on every rank, committed by the DP kernels themselves
            FGR_CHECK_CUDA(g, fgr_launch_dp(g, st, nv, c.exec + o0, nl, n9, cnt - nl - n9 - n2, n2, c.h_maxm[b], nullptr,
                                            nullptr, rec, rec_off, rec_cost, o0, true, &c.prep, c.h_lsplit + 5 * b));
            continue;
        }
        for (int r = emu ? 0 : g->rank; r < (emu ? W : g->rank + 1); r++) {
            fgr_split_batch(cnt, nl, h_epre.data() + o0, g->split_min, r, W, sp);
            if (sp[1] > sp[0])
                FGR_CHECK_CUDA(g, fgr_launch_dp(g, st, nv, c.exec + o0 + sp[0], sp[1] - sp[0], 0, 0, 0, c.h_maxm[b], nullptr,
                                                nullptr, rec, rec_off, rec_cost, o0 + sp[0], false, &c.prep));
            if (sp[3] > sp[2]) {
                // the rank's small chunk [sp2, sp3) crosses the class boundaries nl+n9 and cnt-n2
                const int b1 = nl + n9, b2 = cnt - n2;
                const int cL = max(0, min(sp[3], b1) - sp[2]);
                const int cS = max(0, min(sp[3], b2) - max(sp[2], b1));
                const int cT = sp[3] - sp[2] - cL - cS;
                FGR_CHECK_CUDA(g, fgr_launch_dp(g, st, nv, c.exec + o0 + sp[2], 0, cL, cS, cT, 0, nullptr, nullptr, rec,
                                                rec_off, rec_cost, o0 + sp[2], false, &c.prep));
            }
        }
        g->stats.exchanged_batches++;
        if (!emu) {
            const int ps = fgr_prof_begin(g, PROF_EXCHANGE, st);
            ncclResult_t nr = ncclGroupStart();
            if (nr == ncclSuccess)
                nr = ncclAllReduce(rec + h_roff[b], rec + h_roff[b], (size_t)(h_roff[b + 1] - h_roff[b]), ncclUint32,
                                   ncclSum, g->comm, st);
            if (nr == ncclSuccess)
                nr = ncclAllReduce(rec_cost + o0, rec_cost + o0, (size_t)cnt, ncclUint32, ncclSum, g->comm, st);
            ncclResult_t ne = ncclGroupEnd();
            fgr_prof_end(g, ps, st);
            if (nr != ncclSuccess || ne != ncclSuccess) {
                g->broken = true;
                return fgr_set_error(FGR_ERR_NCCL, "NCCL all-reduce failed: %s",
                                     ncclGetErrorString(nr != ncclSuccess ? nr : ne));
            }
        }
        FGR_CHECK_CUDA(g, fgr_launch_commit(g, st, nv, c.exec + o0, cnt, rec, rec_off, o0));
    }
    if (R > 0) {
        k_scatter_records<<<(unsigned)(((size_t)R * 32 + 255) / 256), 256, 0, st>>>(R, c.exec, nets->node_offset,
                                                                                     rec_off, rec, rec_cost, seg_out,
                                                                                     net_cost);
        FGR_CHECK_CUDA(g, cudaGetLastError());
    }
    FGR_CHECK_CUDA(g, fgr_launch_hyb_zmid(g, st, seg_out, zmid_out));
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_comm_unique_id(void* out128) {
    if (!out128) return fgr_set_error(FGR_ERR_INVALID, "out is NULL");
    ncclUniqueId id;
    ncclResult_t r = ncclGetUniqueId(&id);
    if (r != ncclSuccess) return fgr_set_error(FGR_ERR_NCCL, "ncclGetUniqueId: %s", ncclGetErrorString(r));
    static_assert(sizeof(ncclUniqueId) == 128, "NCCL unique id is 128 bytes");
    memcpy(out128, &id, 128);
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_comm_init(fgr_grid* g, const void* uid, int rank, int world) {
    if (!g || !uid) return fgr_set_error(FGR_ERR_INVALID, "NULL argument");
    if (world < 1 || rank < 0 || rank >= world) return fgr_set_error(FGR_ERR_INVALID, "bad rank/world %d/%d", rank, world);
    if (g->broken) return fgr_set_error(FGR_ERR_STATE, "grid unusable after an earlier CUDA/NCCL error");
    FGR_CHECK_CUDA(g, cudaSetDevice(g->device));
    if (g->comm) { ncclCommDestroy(g->comm); g->comm = nullptr; }
    ncclUniqueId id;
    memcpy(&id, uid, sizeof(id));
    ncclResult_t r = ncclCommInitRank(&g->comm, world, id, rank);
    if (r != ncclSuccess) { g->comm = nullptr; return fgr_set_error(FGR_ERR_NCCL, "ncclCommInitRank: %s", ncclGetErrorString(r)); }
    g->rank = rank;
    g->world = world;
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_run_host(fgr_grid* g, int32_t N, int32_t M, const int32_t* h_off, const int16_t* h_x,
                                           const int16_t* h_y, const int8_t* h_plo, const int8_t* h_phi,
                                           const int32_t* h_par, uint32_t* h_seg, uint32_t* h_cost,
                                           int32_t* h_nb, void* stream) {
    return fgr_run_host_ex(g, N, M, h_off, h_x, h_y, h_plo, h_phi, h_par, h_seg, nullptr, h_cost, h_nb, stream);
}

extern "C" FGR_API fgr_status fgr_run_host_ex(fgr_grid* g, int32_t N, int32_t M, const int32_t* h_off,
                                              const int16_t* h_x, const int16_t* h_y, const int8_t* h_plo,
                                              const int8_t* h_phi, const int32_t* h_par, uint32_t* h_seg,
                                              int32_t* h_zmid, uint32_t* h_cost, int32_t* h_nb, void* stream) {
    if (!g) return fgr_set_error(FGR_ERR_INVALID, "grid is NULL");
    if (g->broken) return fgr_set_error(FGR_ERR_STATE, "grid unusable after an earlier CUDA/NCCL error");
    if (N < 0 || M < 0 || (N > 0 && (!h_off || !h_x || !h_y || !h_plo || !h_phi || !h_par)))
        return fgr_set_error(FGR_ERR_INVALID, "bad host arrays");
    cudaStream_t st = (cudaStream_t)stream;
    FGR_CHECK_CUDA(g, cudaSetDevice(g->device));
    // one device slab: off | par | seg | zmid | batch | order | boff | cost | x | y | plo | phi
    const size_t bytes = 4 * ((size_t)N + 1) + 4 * (size_t)M + 4 * (size_t)M + 4 * (size_t)M + 4 * (size_t)N +
                         4 * (size_t)N + 4 * ((size_t)N + 1) + 4 * (size_t)N + 2 * (size_t)M + 2 * (size_t)M + M + M + 256;
    cudaError_t e;
    char* p = (char*)fgr_scratch(g->s_rec[0], bytes + 64, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "run_host buffers");
    int32_t* d_off = (int32_t*)p; p += 4 * ((size_t)N + 1);
    int32_t* d_par = (int32_t*)p; p += 4 * (size_t)M;
    uint32_t* d_seg = (uint32_t*)p; p += 4 * (size_t)M;
    int32_t* d_zmid = (int32_t*)p; p += 4 * (size_t)M;
    int32_t* d_bat = (int32_t*)p; p += 4 * (size_t)N;
    int32_t* d_ord = (int32_t*)p; p += 4 * (size_t)N;
    int32_t* d_boff = (int32_t*)p; p += 4 * ((size_t)N + 1);
    uint32_t* d_cost = (uint32_t*)p; p += 4 * (size_t)N;
    int16_t* d_x = (int16_t*)p; p += 2 * (size_t)M;
    int16_t* d_y = (int16_t*)p; p += 2 * (size_t)M;
    int8_t* d_plo = (int8_t*)p; p += M;
    int8_t* d_phi = (int8_t*)p;
    FGR_CHECK_CUDA(g, cudaMemcpyAsync(d_off, h_off, 4 * ((size_t)N + 1), cudaMemcpyHostToDevice, st));
    if (M > 0) {
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(d_par, h_par, 4 * (size_t)M, cudaMemcpyHostToDevice, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(d_x, h_x, 2 * (size_t)M, cudaMemcpyHostToDevice, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(d_y, h_y, 2 * (size_t)M, cudaMemcpyHostToDevice, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(d_plo, h_plo, (size_t)M, cudaMemcpyHostToDevice, st));
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(d_phi, h_phi, (size_t)M, cudaMemcpyHostToDevice, st));
    }
    fgr_nets n;
    n.num_nets = N; n.num_nodes = M; n.node_offset = d_off; n.x = d_x; n.y = d_y; n.pin_lo = d_plo; n.pin_hi = d_phi;
    n.parent = d_par;
    fgr_status s = fgr_grid_set_demand(g, nullptr, stream);
    if (s != FGR_OK) return s;
    int32_t B = 0;
    s = fgr_plan(g, &n, d_bat, d_ord, d_boff, &B, stream);
    if (s != FGR_OK) return s;
    s = fgr_route_all_ex(g, &n, d_ord, d_boff, B, d_seg, h_zmid ? d_zmid : nullptr, d_cost, stream);
    if (s != FGR_OK) return s;
    if (h_seg && M > 0) FGR_CHECK_CUDA(g, cudaMemcpyAsync(h_seg, d_seg, 4 * (size_t)M, cudaMemcpyDeviceToHost, st));
    if (h_zmid && M > 0) FGR_CHECK_CUDA(g, cudaMemcpyAsync(h_zmid, d_zmid, 4 * (size_t)M, cudaMemcpyDeviceToHost, st));
    if (h_cost && N > 0) FGR_CHECK_CUDA(g, cudaMemcpyAsync(h_cost, d_cost, 4 * (size_t)N, cudaMemcpyDeviceToHost, st));
    FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));
    if (h_nb) *h_nb = B;
    return FGR_OK;
}
