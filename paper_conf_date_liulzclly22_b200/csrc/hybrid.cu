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

constexpr int kTmThreads = 128;
constexpr int kTmTile = 64;     // candidates whose legs are staged in shared memory at a time

// Transfer matrices M[s][lt][ls] (values) and A[s][lt][ls] (Z argmin mid | lb << 16, 0xFFFFFFFF = the L shape
// or no candidate) of the hybrid edges s = slot0 .. slot0 + gridDim.x - 1, one CTA per edge.
// Per family (HVH: ls, lt horizontal; VHV: ls, lt vertical) the candidates are processed in tiles:
// the CTA first stages the three leg costs of every layer for a tile of bend positions in shared
// memory (each leg one prefix difference), then every thread owns one (ls, lt) entry (or a share of
// one) and scans the tile: value = leg1(ls) + min_lb [V(ls,lb) + leg2(lb) + V(lb,lt)] + leg3(lt)
// (Eqs. (11)-(14)); the running minimum of the packed (value, mid, lb) key is Eq. (10)'s merge.
template <int LT>
__global__ void __launch_bounds__(kTmThreads) k_hyb_tm(GridView g, NetsView nv, const int32_t* __restrict__ hlist,
                                                      const int32_t* __restrict__ hpar, int slot0,
                                                      uint32_t* __restrict__ M, uint32_t* __restrict__ A) {
    __shared__ uint32_t legs[kTmTile][3][LT];
    __shared__ unsigned long long best_s[LT * LT];
    const int s = slot0 + blockIdx.x;
    const int gv = hlist[s], gu = hpar[s];
    const int xv = nv.x[gv], yv = nv.y[gv], xu = nv.x[gu], yu = nv.y[gu];
    const int t = threadIdx.x;
    uint32_t vp[LT];
    int dl[LT], sl[LT];
#pragma unroll
    for (int l = 0; l < LT; l++) { vp[l] = g.viapre[l]; dl[l] = g.dir[l]; sl[l] = g.slot[l]; }
    uint32_t* Ms = M + (size_t)s * LT * LT;
    uint32_t* As = A + (size_t)s * LT * LT;
    const int xlo = min(xv, xu), ylo = min(yv, yu);
    // the L shape for every (ls, lt) of opposite directions (bend 0 if leg 1 is horizontal)
    for (int e = t; e < LT * LT; e += kTmThreads) {
        const int ls = e % LT, lt = e / LT;
        best_s[e] = ~0ull;
        const int dls = g.dir[ls], dlt = g.dir[lt];
        if (dls != dlt) {
            const int sls = g.slot[ls], slt = g.slot[lt];
            const uint32_t l1 = dls == 0 ? leg_of(g.h, yv, xv, xu, sls) : leg_of(g.v, xv, yv, yu, sls);
            const uint32_t l2 = dls == 0 ? leg_of(g.v, xu, yv, yu, slt) : leg_of(g.h, yu, xv, xu, slt);
            const uint32_t vv = g.viapre[max(ls, lt)] - g.viapre[min(ls, lt)];
            Ms[lt * LT + ls] = l1 + vv + l2;
            As[lt * LT + ls] = 0xFFFFFFFFu;
        }
    }
    for (int f = 0; f < 2; f++) {   // f = 0: HVH (ls, lt horizontal), f = 1: VHV
        const int nmid = f == 0 ? abs(xu - xv) - 1 : abs(yu - yv) - 1;
        int nf = 0;
#pragma unroll
        for (int l = 0; l < LT; l++) nf += dl[l] == f ? 1 : 0;
        const int nE = nf * nf;
        if (nmid <= 0 || nE == 0) continue;
        const int tpe = nE <= kTmThreads ? kTmThreads / nE : 1;   // threads sharing one entry
        // this thread's entries (at most 2: nE <= 15 * 15)
        int ls_[2] = {-1, -1}, lt_[2] = {-1, -1};
        uint32_t vsum[2][LT];
        unsigned long long best[2] = {~0ull, ~0ull};
        const int sub = t % tpe;
        for (int k = 0; k < 2; k++) {
            const int e = t / tpe + k * (kTmThreads / tpe);
            if (e >= nE || (k == 1 && tpe > 1)) break;
            int a = e / nf, b = e % nf, ls = -1, lt = -1;
#pragma unroll
            for (int l = 0; l < LT; l++)
                if (dl[l] == f) { if (a == 0) ls = l; if (b == 0) lt = l; a--; b--; }
            ls_[k] = ls; lt_[k] = lt;
            uint32_t vls = 0, vlt = 0;
#pragma unroll
            for (int l = 0; l < LT; l++) { vls = l == ls ? vp[l] : vls; vlt = l == lt ? vp[l] : vlt; }
#pragma unroll
            for (int lb = 0; lb < LT; lb++) {
                const uint32_t a1 = vp[lb] > vls ? vp[lb] - vls : vls - vp[lb];
                const uint32_t a2 = vp[lb] > vlt ? vp[lb] - vlt : vlt - vp[lb];
                vsum[k][lb] = a1 + a2;   // V(ls, lb) + V(lb, lt)
            }
        }
        const int base = f == 0 ? xlo + 1 : ylo + 1;
        for (int c0 = 0; c0 < nmid; c0 += kTmTile) {
            const int nt = min(kTmTile, nmid - c0);
            __syncthreads();
            for (int it = t; it < nt * LT; it += kTmThreads) {
                const int i = it / LT, l = it % LT;
                const int mid = base + c0 + i;
                const int sll = g.slot[l];
                if (g.dir[l] == f) {
                    legs[i][0][l] = f == 0 ? leg_of(g.h, yv, xv, mid, sll) : leg_of(g.v, xv, yv, mid, sll);
                    legs[i][2][l] = f == 0 ? leg_of(g.h, yu, mid, xu, sll) : leg_of(g.v, xu, mid, yu, sll);
                } else {
                    legs[i][1][l] = f == 0 ? leg_of(g.v, mid, yv, yu, sll) : leg_of(g.h, mid, xv, xu, sll);
                }
            }
            __syncthreads();
            for (int k = 0; k < 2; k++) {
                if (ls_[k] < 0) break;
                const int ls = ls_[k], lt = lt_[k];
                for (int i = sub; i < nt; i += tpe) {
                    uint32_t bv = 0xFFFFFFFFu;
                    int blb = 0;
#pragma unroll
                    for (int lb = 0; lb < LT; lb++)
                        if (dl[lb] != f) {
                            const uint32_t c = vsum[k][lb] + legs[i][1][lb];
                            if (c < bv) { bv = c; blb = lb; }   // first minimum: smallest lb (R25)
                        }
                    const uint32_t val = legs[i][0][ls] + bv + legs[i][2][lt];
                    const unsigned long long key =
                        ((unsigned long long)val << 32) | ((unsigned)(base + c0 + i) << 4) | (unsigned)blb;
                    best[k] = key < best[k] ? key : best[k];
                }
            }
        }
        for (int k = 0; k < 2; k++)
            if (ls_[k] >= 0) atomicMin(&best_s[lt_[k] * LT + ls_[k]], best[k]);
    }
    __syncthreads();
    for (int e = t; e < LT * LT; e += kTmThreads) {
        const int ls = e % LT, lt = e / LT;
        if (g.dir[ls] == g.dir[lt]) {
            const unsigned long long k = best_s[lt * LT + ls];
            const bool none = k == ~0ull;
            Ms[lt * LT + ls] = none ? FGR_INF : (uint32_t)(k >> 32);
            As[lt * LT + ls] = none ? 0xFFFFFFFFu : ((uint32_t)((k >> 4) & 0xFFFF) | ((uint32_t)(k & 15) << 16));
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
    k_hyb_tm<LT><<<n, kTmThreads, 0, st>>>(g->view, nv, g->hy.list, g->hy.par, slot0, g->hy.M, g->hy.A);
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
