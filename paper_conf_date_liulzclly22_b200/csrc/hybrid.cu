// hybrid.cu — hybrid L+Z pattern routing (§III-E/F, §IV-D).
//
// A bent tree edge v -> u whose two-pin HPWL |dx|+|dy| lies in [t1, t2] (the
// paper's "medium" two-pin nets, L1240-1298, reading R23) takes the hybrid
// candidate set of L1043-1092: the two L shapes plus every Z shape whose bend
// points lie strictly inside the box (reading R24):
//   HVH (ls, lt horizontal, lb vertical): Bs = (xm, y_v), Bt = (xm, y_u), x_v < xm < x_u
//   VHV (ls, lt vertical, lb horizontal): Bs = (x_v, ym), Bt = (x_u, ym), y_v < ym < y_u
// with Eq. (8) c = cw(Ps,Bs,ls) + cv(Bs,ls,lb) + cw(Bs,Bt,lb) + cv(Bt,lb,lt) + cw(Bt,Pt,lt)
// (L831-842) and the candidate flows of Eqs. (11)-(14) merged by Eq. (10) (L864-1032).
//
// B200 mapping.  Costs are fixed during a batch, so the whole candidate set of
// an edge folds into one L x L transfer matrix, independent of the tree DP:
//     M_e(ls, lt) = min over candidates c and lb of [legs + bend vias](c, ls, lb, lt)
// and the tree DP's edge step becomes E_v(lt) = min_ls [B_v(ls) + M_e(ls, lt)]
// (the same min-plus vector x matrix product as the L edge step).  k_hyb_tm
// computes M_e for every hybrid edge of a batch right after the cost refresh:
// one CTA per edge, warp w owns the departure layers ls = w, w+4, ..., its lanes
// stride over the candidate bend positions (the M+N candidate flows of Fig. 10
// in parallel), and a warp min-reduction of packed (value, mid, lb) keys is the
// merge step of Eq. (10) with reading R25's tie order.  For (ls, lt) of opposite
// directions the only candidate is the L shape; for equal directions only Z
// shapes apply, so L and Z never tie inside one matrix entry.
#include <cub/cub.cuh>

#include "fgr_internal.cuh"

namespace {

__device__ __forceinline__ uint32_t prefix_at(const DirView& d, int line, int pos, int sl) {
    return d.SB[((size_t)line * d.nseg + (pos >> FGR_SEG_SHIFT)) * d.W + sl] + d.P[((size_t)line * d.len + pos) * d.W + sl];
}

// wire cost of the leg [a, b] (either order) on `line` in layer slot sl: difference of two prefixes (R19)
__device__ __forceinline__ uint32_t leg_of(const DirView& d, int line, int a, int b, int sl) {
    const int lo = min(a, b), hi = max(a, b);
    return prefix_at(d, line, hi, sl) - prefix_at(d, line, lo, sl);
}

__device__ __forceinline__ bool hyb_edge(int xv, int yv, int xu, int yu, int t1, int t2) {
    if (xv == xu || yv == yu) return false;
    const int h = abs(xv - xu) + abs(yv - yu);
    return h >= t1 && h <= t2;
}

// one warp per net (exec position r): count its hybrid edges
__global__ void k_hyb_count(int R, const int32_t* __restrict__ exec, NetsView nv, int t1, int t2, int32_t* __restrict__ cnt) {
    const int r = (int)((blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5);
    if (r >= R) return;
    const int net = exec[r];
    const int a0 = nv.off[net], m = nv.off[net + 1] - a0;
    int c = 0;
    for (int i = 1 + lane_id(); i < m; i += 32) {
        const int u = a0 + nv.par[a0 + i];
        c += hyb_edge(nv.x[a0 + i], nv.y[a0 + i], nv.x[u], nv.y[u], t1, t2) ? 1 : 0;
    }
    c = __reduce_add_sync(0xffffffffu, c);
    if (lane_id() == 0) cnt[r] = c;
}

// one warp per net: slots in node order from the net's base; zmid of its nodes reset to -1
__global__ void k_hyb_fill(int R, const int32_t* __restrict__ exec, NetsView nv, int t1, int t2,
                           const int32_t* __restrict__ base, int32_t* __restrict__ hnet, int32_t* __restrict__ hslot,
                           int32_t* __restrict__ hlist, int32_t* __restrict__ hpar, int32_t* __restrict__ zmid) {
    const int r = (int)((blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5);
    if (r >= R) return;
    const int lane = lane_id();
    const int net = exec[r];
    const int a0 = nv.off[net], m = nv.off[net + 1] - a0;
    const int b0 = base[r], n = base[r + 1] - b0;
    if (lane == 0) hnet[net] = n > 0 ? b0 : -1;
    if (zmid)
        for (int i = lane; i < m; i += 32) zmid[a0 + i] = -1;
    if (n == 0) return;
    int k = b0;
    for (int c0 = 0; c0 < m; c0 += 32) {
        const int i = c0 + lane;
        bool hy = false;
        int u = 0;
        if (i >= 1 && i < m) {
            u = a0 + nv.par[a0 + i];
            hy = hyb_edge(nv.x[a0 + i], nv.y[a0 + i], nv.x[u], nv.y[u], t1, t2);
        }
        const unsigned b = __ballot_sync(0xffffffffu, hy);
        if (i < m) {
            const int s = hy ? k + __popc(b & ((1u << lane) - 1u)) : -1;
            hslot[a0 + i] = s;
            if (hy) { hlist[s] = a0 + i; hpar[s] = u; }
        }
        k += __popc(b);
    }
}

__global__ void k_hyb_boff(int n, const int32_t* __restrict__ boff, const int32_t* __restrict__ base, int32_t* __restrict__ out) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) out[i] = base[boff[i]];
}

constexpr int kTmWarps = 4;

// Transfer matrices M[s][lt][ls] (values) and A[s][lt][ls] (Z argmin mid | lb << 16, 0xFFFFFFFF = the L shape
// or no candidate) of the hybrid edges s = slot0 .. slot0 + gridDim.x - 1.
template <int LT>
__global__ void __launch_bounds__(32 * kTmWarps) k_hyb_tm(GridView g, NetsView nv, const int32_t* __restrict__ hlist,
                                                         const int32_t* __restrict__ hpar, int slot0,
                                                         uint32_t* __restrict__ M, uint32_t* __restrict__ A) {
    const int s = slot0 + blockIdx.x;
    const int gv = hlist[s], gu = hpar[s];
    const int xv = nv.x[gv], yv = nv.y[gv], xu = nv.x[gu], yu = nv.y[gu];
    const int warp = threadIdx.x >> 5, lane = lane_id();
    uint32_t vp[LT];
    int dl[LT], sl[LT];
#pragma unroll
    for (int l = 0; l < LT; l++) { vp[l] = g.viapre[l]; dl[l] = g.dir[l]; sl[l] = g.slot[l]; }
    auto via = [&](int a, int b) -> uint32_t {   // V(min, max) for compile-time-unrolled indices
        return vp[a] > vp[b] ? vp[a] - vp[b] : vp[b] - vp[a];
    };
    uint32_t* Ms = M + (size_t)s * LT * LT;
    uint32_t* As = A + (size_t)s * LT * LT;
#pragma unroll
    for (int ls = 0; ls < LT; ls++) {
        if (ls % kTmWarps != warp) continue;
        const int dls = dl[ls];
        // the L shape for every lt of the other direction (bend 0 if leg 1 is horizontal)
#pragma unroll
        for (int lt = 0; lt < LT; lt++)
            if (lane == lt && dl[lt] != dls) {
                const uint32_t l1 = dls == 0 ? leg_of(g.h, yv, xv, xu, sl[ls]) : leg_of(g.v, xv, yv, yu, sl[ls]);
                const uint32_t l2 = dls == 0 ? leg_of(g.v, xu, yv, yu, sl[lt]) : leg_of(g.h, yu, xv, xu, sl[lt]);
                Ms[lt * LT + ls] = l1 + via(ls, lt) + l2;
                As[lt * LT + ls] = 0xFFFFFFFFu;
            }
        // Z shapes (lt in the direction of ls): candidate flows over the interior bend positions
        const bool hvh = dls == 0;
        const int p0 = hvh ? min(xv, xu) + 1 : min(yv, yu) + 1;
        const int p1 = hvh ? max(xv, xu) - 1 : max(yv, yu) - 1;
        unsigned long long best[LT];
#pragma unroll
        for (int lt = 0; lt < LT; lt++) best[lt] = ~0ull;
        for (int mid = p0 + lane; mid <= p1; mid += 32) {
            // Eq. (11): leg 1 on ls;  Eq. (12): bend via + leg 2 on lb;  Eq. (13): bend via + leg 3 on lt
            const uint32_t w1 = hvh ? leg_of(g.h, yv, xv, mid, sl[ls]) : leg_of(g.v, xv, yv, mid, sl[ls]);
            uint32_t t2v[LT];
#pragma unroll
            for (int lb = 0; lb < LT; lb++)
                if (dl[lb] != dls)
                    t2v[lb] = via(ls, lb) + (hvh ? leg_of(g.v, mid, yv, yu, sl[lb]) : leg_of(g.h, mid, xv, xu, sl[lb]));
#pragma unroll
            for (int lt = 0; lt < LT; lt++)
                if (dl[lt] == dls) {
                    uint32_t bv = 0xFFFFFFFFu;
                    int blb = 0;
#pragma unroll
                    for (int lb = 0; lb < LT; lb++)
                        if (dl[lb] != dls) {
                            const uint32_t c = t2v[lb] + via(lb, lt);
                            if (c < bv) { bv = c; blb = lb; }   // first minimum: smallest lb (R25)
                        }
                    const uint32_t w3 = hvh ? leg_of(g.h, yu, mid, xu, sl[lt]) : leg_of(g.v, xu, mid, yu, sl[lt]);
                    const unsigned long long key =
                        ((unsigned long long)(w1 + bv + w3) << 32) | ((unsigned)mid << 4) | (unsigned)blb;
                    best[lt] = key < best[lt] ? key : best[lt];
                }
        }
        // merge step, Eq. (10): warp minimum of the packed (value, mid, lb) keys
#pragma unroll
        for (int lt = 0; lt < LT; lt++)
            if (dl[lt] == dls) {
                unsigned long long k = best[lt];
#pragma unroll
                for (int off = 16; off; off >>= 1) {
                    const unsigned long long o = __shfl_xor_sync(0xffffffffu, k, off);
                    k = o < k ? o : k;
                }
                if (lane == 0) {
                    const bool none = k == ~0ull;
                    Ms[lt * LT + ls] = none ? FGR_INF : (uint32_t)(k >> 32);
                    As[lt * LT + ls] = none ? 0xFFFFFFFFu : ((uint32_t)((k >> 4) & 0xFFFF) | ((uint32_t)(k & 15) << 16));
                }
            }
    }
}

// zmid[node] of the Z routes chosen (seg bend 2 / 3)
__global__ void k_hyb_zmid(int n, int L, const int32_t* __restrict__ hlist, const uint32_t* __restrict__ seg,
                           const uint32_t* __restrict__ A, int32_t* __restrict__ zmid) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= n) return;
    const int gv = hlist[s];
    const uint32_t sg = seg[gv];
    if ((sg & 0xFF) >= 2 && sg != 0xFFFFFFFFu) {
        const int ls = (sg >> 8) & 0xFF, lt = (sg >> 16) & 0xFF;
        zmid[gv] = (int32_t)A[((size_t)s * L + lt) * L + ls];
    }
}

template <int LT>
cudaError_t launch_tm_lt(fgr_grid* g, cudaStream_t st, const NetsView& nv, int slot0, int n) {
    k_hyb_tm<LT><<<n, 32 * kTmWarps, 0, st>>>(g->view, nv, g->hy.list, g->hy.par, slot0, g->hy.M, g->hy.A);
    return cudaGetLastError();
}

}  // namespace

// Per-stage hybrid tables for the nets exec[0..R): slots in exec order (so the
// slots of one batch are contiguous when exec is batch-major), per-batch slot
// offsets on the host (boff = the batch offsets into exec, nb batches; NULL = one
// batch), zmid of the listed nets reset to -1.  One sync.
fgr_status fgr_hyb_prepare(fgr_grid* g, cudaStream_t st, const NetsView& nv, int num_nets, int num_nodes,
                           const int32_t* exec, int R, const int32_t* boff, int nb, int32_t* zmid) {
    HybState& h = g->hy;
    h.active = false;
    h.nslots = 0;
    if (g->hyb_t1 > g->hyb_t2 || R == 0) return FGR_OK;
    cudaError_t e;
    int32_t* cnt = (int32_t*)fgr_scratch(g->s_hyb[0], sizeof(int32_t) * (2 * ((size_t)R + 1) + (size_t)nb + 1) + 64, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "hybrid counts");
    int32_t* base = cnt + R + 1;
    int32_t* dboff = base + R + 1;
    const unsigned blocks = (unsigned)(((size_t)R * 32 + 255) / 256);
    k_hyb_count<<<blocks, 256, 0, st>>>(R, exec, nv, g->hyb_t1, g->hyb_t2, cnt);
    FGR_CHECK_CUDA(g, cudaGetLastError());
    FGR_CHECK_CUDA(g, cudaMemsetAsync(cnt + R, 0, sizeof(int32_t), st));
    size_t tb = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt, base, R + 1, st);
    void* tmp = fgr_scratch(g->s_hyb[1], tb, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "hybrid scan scratch");
    FGR_CHECK_CUDA(g, cub::DeviceScan::ExclusiveSum(tmp, tb, cnt, base, R + 1, st));
    int total = 0;
    FGR_CHECK_CUDA(g, cudaMemcpyAsync(&total, base + R, sizeof(int), cudaMemcpyDeviceToHost, st));
    FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));
    const size_t L2 = (size_t)g->L * g->L;
    const size_t bytes = sizeof(int32_t) * ((size_t)num_nets + (size_t)num_nodes + 2 * (size_t)total) +
                         sizeof(uint32_t) * 2 * L2 * (size_t)total + 6 * 256;
    char* p = (char*)fgr_scratch(g->s_hyb[2], bytes, &e);
    if (e != cudaSuccess) return fgr_cuda_fail(g, e, "hybrid tables");
    auto take = [&](size_t n) { char* q = p; p += (n + 255) & ~(size_t)255; return q; };
    h.net = (int32_t*)take(sizeof(int32_t) * (size_t)num_nets);
    h.slot = (int32_t*)take(sizeof(int32_t) * (size_t)num_nodes);
    h.list = (int32_t*)take(sizeof(int32_t) * (size_t)total);
    h.par = (int32_t*)take(sizeof(int32_t) * (size_t)total);
    h.M = (uint32_t*)take(sizeof(uint32_t) * L2 * (size_t)total);
    h.A = (uint32_t*)take(sizeof(uint32_t) * L2 * (size_t)total);
    if (num_nets > 0) FGR_CHECK_CUDA(g, cudaMemsetAsync(h.net, 0xFF, sizeof(int32_t) * (size_t)num_nets, st));
    k_hyb_fill<<<blocks, 256, 0, st>>>(R, exec, nv, g->hyb_t1, g->hyb_t2, base, h.net, h.slot, h.list, h.par, zmid);
    FGR_CHECK_CUDA(g, cudaGetLastError());
    h.nslots = total;
    h.active = total > 0;
    h.boff.assign(nb + 1, 0);
    if (boff && nb > 0) {
        k_hyb_boff<<<(nb + 1 + 255) / 256, 256, 0, st>>>(nb + 1, boff, base, dboff);
        FGR_CHECK_CUDA(g, cudaGetLastError());
        FGR_CHECK_CUDA(g, cudaMemcpyAsync(h.boff.data(), dboff, sizeof(int32_t) * (nb + 1), cudaMemcpyDeviceToHost, st));
        FGR_CHECK_CUDA(g, cudaStreamSynchronize(st));
    } else {
        h.boff[0] = 0;
        h.boff[nb] = total;
    }
    return FGR_OK;
}

cudaError_t fgr_launch_hyb_tm(fgr_grid* g, cudaStream_t st, const NetsView& nv, int slot0, int n) {
    if (n <= 0 || !g->hy.active) return cudaSuccess;
    const int ps = fgr_prof_begin(g, PROF_HYBRID, st);
    cudaError_t e;
    switch (g->L) {
#define FGR_LT(k) case k: e = launch_tm_lt<k>(g, st, nv, slot0, n); break;
        FGR_LT(2) FGR_LT(3) FGR_LT(4) FGR_LT(5) FGR_LT(6) FGR_LT(7) FGR_LT(8) FGR_LT(9) FGR_LT(10) FGR_LT(11)
        FGR_LT(12) FGR_LT(13) FGR_LT(14) FGR_LT(15) FGR_LT(16)
#undef FGR_LT
        default: e = cudaErrorInvalidValue;
    }
    fgr_prof_end(g, ps, st);
    g->stats.kernel_launches++;
    return e;
}

cudaError_t fgr_launch_hyb_zmid(fgr_grid* g, cudaStream_t st, const uint32_t* seg, int32_t* zmid) {
    if (!zmid || !g->hy.active) return cudaSuccess;
    const int n = g->hy.nslots;
    k_hyb_zmid<<<(n + 255) / 256, 256, 0, st>>>(n, g->L, g->hy.list, seg, g->hy.A, zmid);
    g->stats.kernel_launches++;
    return cudaGetLastError();
}
