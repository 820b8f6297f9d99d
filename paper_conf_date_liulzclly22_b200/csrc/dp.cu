// dp.cu — S4 tree DP + S5 backtrack + S6 commit.
//
// Per net (§III-D), for every tree edge v -> u (v = child =
// source Ps, u = parent = target Pt, L566-571):
//   Eq. (1)  c(P{Ps,B_ls,T_lt}) = cw(Ps,B,ls) + cv(B,ls,lt) + cw(B,Tlt,lt)     L594-608
//   Eq. (2)  cbc(Ps,ls) = min_{l1..lc} [cv(Ps,ls,l1..lc) + sum_i c*(child_i,li)] L610-645
//            computed exactly by enumerating via spans [lo,hi] (reading R3):
//            F_v(lo,hi) = V(lo,hi) + sum_c min_{l in [lo,hi]} E_c(l)
//            B_v(ls)    = min over spans containing ls and v's pin span of F_v
//   Eqs. (3),(5)-(7)  E_v(lt) = min_ls [w1(ls) + W2(ls,lt)],  w1 = B_v + leg 1,
//            W2 = bend via + leg 2 — a min-plus vector x matrix product         L646-667, L698-756
//   Eq. (4)  root: min over spans containing the root pin span of F_r (R9)      L669-696
// then a top-down backtrack (S5) and the +1 demand commit of every chosen leg
// (S6) with dirty-segment marking for the next cost refresh.
//
// B200 mapping: one warp per net (<= 32 nodes) or one 256-thread CTA per net
// (larger nets); nodes are processed level by level, children before parents
// (the DFS order of PAPER.md L320-333 generalised to a level order); all prefix
// gathers of a net are issued up front (costs are fixed during the DP); the
// per-node tables live in shared memory; every min-plus step is a DPX
// VIADDMNMX (sat_add).  Tie-breaks follow reading R11 exactly.
#include "fgr_internal.cuh"

namespace {

struct Hdr {                  // per-block constants copied to shared memory
    uint32_t viapre[FGR_MAXL + 1];
    uint8_t dir[FGR_MAXL];
    uint8_t slot[FGR_MAXL];
    uint8_t los[2][FGR_MAXL];
};

struct Tabs {
    uint32_t* E;      // [m][L]  E_v(lt) = c*(v -> parent, lt)
    uint32_t* legH;   // [m][2][nH]  0: row y_v, 1: row y_u   (x_v..x_u)
    uint32_t* legV;   // [m][2][nV]  0: col x_v, 1: col x_u   (y_v..y_u)
    uint32_t* cmask;  // warp path: children bitmask [32]
    int16_t* x;
    int16_t* y;
    int16_t* par;
    uint16_t* depth;
    uint16_t* cstart; // CTA path: child CSR [m+1]
    uint16_t* clist;  // CTA path: [m]
    uint16_t* anc;    // CTA path: pointer-jumping scratch [m]
    int8_t* plo;
    int8_t* phi;
    uint8_t* span;    // chosen via span (lo << 4) | hi  (low byte of the packed (value, lo, hi) key)
    uint8_t* recE;    // [m][L] argmin ls of E_v(lt)
    uint8_t* recB;    // [m][L] argmin span of B_v(ls)
};

struct WScr {          // warp-private scratch
    uint32_t* F;      // [L][L]
    uint32_t* B;      // [L]
};

__host__ __device__ inline size_t a16(size_t b) { return (b + 15) & ~(size_t)15; }

__host__ __device__ inline size_t tabs_bytes(int m, int L, int nH, int nV, bool cta) {
    size_t b = 0;
    b += a16((size_t)m * L * 4);
    b += a16((size_t)m * 2 * nH * 4);
    b += a16((size_t)m * 2 * nV * 4);
    if (!cta) b += a16((size_t)m * 4);
    b += 4 * a16((size_t)m * 2);
    if (cta) b += a16((size_t)(m + 1) * 2) + 2 * a16((size_t)m * 2);
    b += 3 * a16((size_t)m);
    b += 2 * a16((size_t)m * L);
    return b;
}

__host__ __device__ inline size_t wscr_bytes(int L) { return a16((size_t)L * L * 4) + a16((size_t)L * 4); }

__device__ inline Tabs carve_tabs(unsigned char* p, int m, int L, int nH, int nV, bool cta) {
    Tabs t;
    t.E = (uint32_t*)p; p += a16((size_t)m * L * 4);
    t.legH = (uint32_t*)p; p += a16((size_t)m * 2 * nH * 4);
    t.legV = (uint32_t*)p; p += a16((size_t)m * 2 * nV * 4);
    t.cmask = nullptr;
    if (!cta) { t.cmask = (uint32_t*)p; p += a16((size_t)m * 4); }
    t.x = (int16_t*)p; p += a16((size_t)m * 2);
    t.y = (int16_t*)p; p += a16((size_t)m * 2);
    t.par = (int16_t*)p; p += a16((size_t)m * 2);
    t.depth = (uint16_t*)p; p += a16((size_t)m * 2);
    t.cstart = t.clist = t.anc = nullptr;
    if (cta) {
        t.cstart = (uint16_t*)p; p += a16((size_t)(m + 1) * 2);
        t.clist = (uint16_t*)p; p += a16((size_t)m * 2);
        t.anc = (uint16_t*)p; p += a16((size_t)m * 2);
    }
    t.plo = (int8_t*)p; p += a16((size_t)m);
    t.phi = (int8_t*)p; p += a16((size_t)m);
    t.span = (uint8_t*)p; p += a16((size_t)m);
    t.recE = p; p += a16((size_t)m * L);
    t.recB = p; p += a16((size_t)m * L);
    return t;
}

__device__ inline WScr carve_wscr(unsigned char* p, int L) {
    WScr w;
    w.F = (uint32_t*)p;
    w.B = (uint32_t*)(p + a16((size_t)L * L * 4));
    return w;
}

__device__ inline void init_hdr(Hdr* h, const GridView& g) {
    for (int i = threadIdx.x; i <= FGR_MAXL; i += blockDim.x) h->viapre[i] = g.viapre[i];
    for (int i = threadIdx.x; i < FGR_MAXL; i += blockDim.x) {
        h->dir[i] = g.dir[i];
        h->slot[i] = g.slot[i];
        h->los[0][i] = g.layer_of_slot[0][i];
        h->los[1][i] = g.layer_of_slot[1][i];
    }
}

struct Out {
    uint32_t* seg;        // [num_nodes] by global node index (direct mode)
    uint32_t* cost;       // [num_nets] by net id (direct mode)
    uint32_t* rec_seg;    // record mode: rec_seg[rec_off[list_base + idx] + local]
    const int32_t* rec_off;
    uint32_t* rec_cost;   // record mode: rec_cost[list_base + idx]
    int list_base;
};

// ------------------------------------------------------------- leg gathers
// Cost of the leg from position a to b (a < b) on `line` for every slot:
// (SB[seg(b)] + P[b]) - (SB[seg(a)] + P[a]), exact in uint32 (R19).
__device__ __forceinline__ void leg_cost(const DirView& d, int line, int a, int b, uint32_t* out) {
    const size_t pa = ((size_t)line * d.len + a) * d.W, pb = ((size_t)line * d.len + b) * d.W;
    const size_t sa = ((size_t)line * d.nseg + (a >> FGR_SEG_SHIFT)) * d.W;
    const size_t sb = ((size_t)line * d.nseg + (b >> FGR_SEG_SHIFT)) * d.W;
    const int nq = d.W >> 2;
#pragma unroll
    for (int q = 0; q < 4; q++) {
        if (q < nq) {
            uint4 Pa = __ldg(reinterpret_cast<const uint4*>(d.P + pa) + q);
            uint4 Pb = __ldg(reinterpret_cast<const uint4*>(d.P + pb) + q);
            uint4 Sa = __ldg(reinterpret_cast<const uint4*>(d.SB + sa) + q);
            uint4 Sb = __ldg(reinterpret_cast<const uint4*>(d.SB + sb) + q);
            uint32_t r[4] = {(Sb.x + Pb.x) - (Sa.x + Pa.x), (Sb.y + Pb.y) - (Sa.y + Pa.y),
                             (Sb.z + Pb.z) - (Sa.z + Pa.z), (Sb.w + Pb.w) - (Sa.w + Pa.w)};
#pragma unroll
            for (int k = 0; k < 4; k++)
                if (4 * q + k < d.cnt) out[4 * q + k] = r[k];
        }
    }
}

// task = 4*(i-1) + type for node i >= 1: 0 = H row y_v, 1 = H row y_u, 2 = V col x_v, 3 = V col x_u
__device__ __forceinline__ void gather_task(const GridView& g, const Tabs& t, int task) {
    const int i = 1 + (task >> 2), type = task & 3;
    const int u = t.par[i];
    const int xv = t.x[i], yv = t.y[i], xu = t.x[u], yu = t.y[u];
    const bool sh = (yv == yu), sv = (xv == xu);
    if ((sh && type != 0) || (sv && type != 2)) return;
    const int nH = g.h.cnt, nV = g.v.cnt;
    if (type < 2) {
        const int row = type == 0 ? yv : yu;
        leg_cost(g.h, row, min(xv, xu), max(xv, xu), t.legH + ((size_t)i * 2 + type) * nH);
    } else {
        const int col = type == 2 ? xv : xu;
        leg_cost(g.v, col, min(yv, yu), max(yv, yu), t.legV + ((size_t)i * 2 + (type - 2)) * nV);
    }
}

// ------------------------------------------------------------- DP steps (one warp)
// F_v(lo,hi) for all spans (lane = lo), then B_v(ls) (lane = ls) or the root minimum.
template <bool CTA>
__device__ __forceinline__ void span_table(const Hdr* h, const Tabs& t, const WScr& w, int v, int L) {
    const int lane = lane_id();
    if (lane < L) {
        uint32_t acc[FGR_MAXL];
        const uint32_t vlo = h->viapre[lane];
#pragma unroll
        for (int hi = 0; hi < FGR_MAXL; hi++) acc[hi] = (hi < L && hi >= lane) ? h->viapre[hi] - vlo : FGR_INF;
        if (CTA) {
            const int c0 = t.cstart[v], c1 = t.cstart[v + 1];
            for (int k = c0; k < c1; k++) {
                const uint32_t* Ec = t.E + (size_t)t.clist[k] * L;
                uint32_t run = FGR_INF;
#pragma unroll
                for (int hi = 0; hi < FGR_MAXL; hi++)
                    if (hi < L && hi >= lane) { run = min(run, Ec[hi]); acc[hi] = sat_add(acc[hi], run); }
            }
        } else {
            uint32_t cm = t.cmask[v];
            while (cm) {
                const int c = __ffs(cm) - 1;
                cm &= cm - 1;
                const uint32_t* Ec = t.E + (size_t)c * L;
                uint32_t run = FGR_INF;
#pragma unroll
                for (int hi = 0; hi < FGR_MAXL; hi++)
                    if (hi < L && hi >= lane) { run = min(run, Ec[hi]); acc[hi] = sat_add(acc[hi], run); }
            }
        }
#pragma unroll
        for (int hi = 0; hi < FGR_MAXL; hi++)
            if (hi < L && hi >= lane) w.F[lane * L + hi] = acc[hi];
    }
    __syncwarp();
}

// Eq. (2) per ls, with the (value, lo, hi) lexicographic tie-break of R11 as one 64-bit min.
__device__ __forceinline__ void node_table(const Tabs& t, const WScr& w, int v, int L) {
    const int lane = lane_id();
    if (lane < L) {
        int a = lane, b = lane;
        const int plo = t.plo[v], phi = t.phi[v];
        if (plo >= 0) { a = min(a, plo); b = max(b, phi); }
        unsigned long long best = ~0ull;
        for (int lo = 0; lo <= a; lo++)
            for (int hi = b; hi < L; hi++) {
                unsigned long long key = ((unsigned long long)w.F[lo * L + hi] << 8) | (unsigned)(lo << 4) | (unsigned)hi;
                best = key < best ? key : best;
            }
        w.B[lane] = (uint32_t)(best >> 8);
        t.recB[(size_t)v * L + lane] = (uint8_t)(best & 0xFF);
    }
    __syncwarp();
}

// Eqs. (1),(3),(5)-(7): E_v(lt) = min_ls [B_v(ls) + leg1(ls) + V(ls,lt) + leg2(lt)], lane = lt.
__device__ __forceinline__ void edge_table(const Hdr* h, const Tabs& t, const WScr& w, int v, int L, int nH, int nV) {
    const int lane = lane_id();
    if (lane < L) {
        const int lt = lane;
        const int u = t.par[v];
        const int xv = t.x[v], yv = t.y[v], xu = t.x[u], yu = t.y[u];
        const int dlt = h->dir[lt];
        uint32_t best = FGR_INF;
        int bls = lt;
        if (yv == yu || xv == xu) {               // straight: one leg on ls = lt (R7)
            const int de = (yv == yu) ? 0 : 1;
            if (dlt == de) {
                const uint32_t leg = de == 0 ? t.legH[(size_t)v * 2 * nH + h->slot[lt]]
                                             : t.legV[(size_t)v * 2 * nV + h->slot[lt]];
                best = sat_add(w.B[lt], leg);
            }
        } else if (dlt == 1) {                    // bend 0: leg 1 H on row y_v, leg 2 V on col x_u
            const uint32_t leg2 = t.legV[((size_t)v * 2 + 1) * nV + h->slot[lt]];
            const uint32_t* l1 = t.legH + (size_t)v * 2 * nH;
            for (int s = 0; s < nH; s++) {
                const int ls = h->los[0][s];
                const uint32_t via = ls < lt ? h->viapre[lt] - h->viapre[ls] : h->viapre[ls] - h->viapre[lt];
                const uint32_t c = sat_add(sat_add(sat_add(w.B[ls], l1[s]), via), leg2);
                if (c < best) { best = c; bls = ls; }
            }
        } else {                                  // bend 1: leg 1 V on col x_v, leg 2 H on row y_u
            const uint32_t leg2 = t.legH[((size_t)v * 2 + 1) * nH + h->slot[lt]];
            const uint32_t* l1 = t.legV + (size_t)v * 2 * nV;
            for (int s = 0; s < nV; s++) {
                const int ls = h->los[1][s];
                const uint32_t via = ls < lt ? h->viapre[lt] - h->viapre[ls] : h->viapre[ls] - h->viapre[lt];
                const uint32_t c = sat_add(sat_add(sat_add(w.B[ls], l1[s]), via), leg2);
                if (c < best) { best = c; bls = ls; }
            }
        }
        t.E[(size_t)v * L + lt] = best;
        t.recE[(size_t)v * L + lt] = (uint8_t)bls;
    }
    __syncwarp();
}

// Generalised Eq. (4): min over spans containing the root pin span; returns the packed key.
__device__ __forceinline__ unsigned long long root_min(const Tabs& t, const WScr& w, int L) {
    const int lane = lane_id();
    unsigned long long best = ~0ull;
    if (lane < L) {
        const int plo = t.plo[0], phi = t.phi[0];
        const int a = plo >= 0 ? plo : L - 1;     // Steiner root: any span
        const int b = plo >= 0 ? phi : 0;
        if (lane <= a)
            for (int hi = max(lane, b); hi < L; hi++) {
                unsigned long long key = ((unsigned long long)w.F[lane * L + hi] << 8) | (unsigned)(lane << 4) | (unsigned)hi;
                best = key < best ? key : best;
            }
    }
#pragma unroll
    for (int off = 16; off; off >>= 1) {
        unsigned long long o = __shfl_xor_sync(0xffffffffu, best, off);
        best = o < best ? o : best;
    }
    return best;
}

// S5: child layer = smallest l in the parent's span minimising E_v(l) (R11).
__device__ __forceinline__ uint32_t backtrack_node(const Hdr* h, const Tabs& t, int v, int L) {
    const int u = t.par[v];
    const int sp = t.span[u];
    const int lo = sp >> 4, hi = sp & 15;
    int lt = lo;
    uint32_t be = t.E[(size_t)v * L + lo];
    for (int l = lo + 1; l <= hi; l++) {
        const uint32_t e = t.E[(size_t)v * L + l];
        if (e < be) { be = e; lt = l; }
    }
    const int ls = t.recE[(size_t)v * L + lt];
    t.span[v] = t.recB[(size_t)v * L + ls];
    const bool straight = (t.x[v] == t.x[u]) || (t.y[v] == t.y[u]);
    const uint32_t bend = straight ? 0u : (h->dir[lt] == 1 ? 0u : 1u);
    return bend | ((uint32_t)ls << 8) | ((uint32_t)lt << 16) | ((uint32_t)straight << 24);
}

// S6: +1 on every unit edge of a leg, and mark the touched segments dirty.
__device__ __forceinline__ void commit_leg(const GridView& g, const DirView& d, int line, int a, int b, int sl) {
    if (a >= b) return;
    int32_t* D = d.D + (size_t)line * d.len * d.W + sl;
    for (int p = a; p < b; p++) atomicAdd(D + (size_t)p * d.W, 1);
    const int s0 = a >> FGR_SEG_SHIFT, s1 = (b - 1) >> FGR_SEG_SHIFT;
    for (int s = s0; s <= s1; s++) {
        const int gs = d.seg_base + line * d.nseg + s;
        if (atomicExch(&g.dseg[gs], 1u) == 0u) {
            const int k = atomicAdd(g.segcount, 1);
            g.seglist[k] = gs;
            atomicAdd(&g.linecnt[d.line_base + line], 1u);
        }
    }
}

__device__ __forceinline__ void commit_edge(const GridView& g, const Hdr* h, int xv, int yv, int xu, int yu, uint32_t seg) {
    const int bend = seg & 0xFF, ls = (seg >> 8) & 0xFF, lt = (seg >> 16) & 0xFF, straight = (seg >> 24) & 0xFF;
    if (straight) {
        if (yv == yu) commit_leg(g, g.h, yv, min(xv, xu), max(xv, xu), h->slot[lt]);
        else commit_leg(g, g.v, xv, min(yv, yu), max(yv, yu), h->slot[lt]);
        return;
    }
    if (bend == 0) {   // H on row y_v (layer ls), V on col x_u (layer lt)
        commit_leg(g, g.h, yv, min(xv, xu), max(xv, xu), h->slot[ls]);
        commit_leg(g, g.v, xu, min(yv, yu), max(yv, yu), h->slot[lt]);
    } else {           // V on col x_v (layer ls), H on row y_u (layer lt)
        commit_leg(g, g.v, xv, min(yv, yu), max(yv, yu), h->slot[ls]);
        commit_leg(g, g.h, yu, min(xv, xu), max(xv, xu), h->slot[lt]);
    }
}

// ------------------------------------------------------------- kernels
// Warp path: one warp per net with <= 32 nodes.
__global__ void __launch_bounds__(FGR_CTA_THREADS) k_dp_small(GridView g, NetsView nv, const int32_t* __restrict__ list,
                                                               int count, Out o, int commit, int32_t* reset_ptr) {
    extern __shared__ __align__(16) unsigned char smem[];
    Hdr* h = reinterpret_cast<Hdr*>(smem);
    init_hdr(h, g);
    if (reset_ptr && blockIdx.x == 0 && threadIdx.x == 0) *reset_ptr = 0;
    __syncthreads();
    const int L = g.L, nH = g.h.cnt, nV = g.v.cnt;
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int idx = blockIdx.x * FGR_WARPS_PER_CTA + warp;
    if (idx >= count) return;
    const size_t per_warp = a16(sizeof(Hdr)) ;
    unsigned char* base = smem + per_warp + (size_t)warp * (tabs_bytes(32, L, nH, nV, false) + wscr_bytes(L));
    Tabs t = carve_tabs(base, 32, L, nH, nV, false);
    WScr w = carve_wscr(base + tabs_bytes(32, L, nH, nV, false), L);
    const int net = list[idx];
    const int a0 = nv.off[net];
    const int m = nv.off[net + 1] - a0;
    // node data (lane = node)
    int par = -1, xx = 0, yy = 0;
    if (lane < m) {
        xx = nv.x[a0 + lane]; yy = nv.y[a0 + lane]; par = nv.par[a0 + lane];
        t.x[lane] = (int16_t)xx; t.y[lane] = (int16_t)yy; t.par[lane] = (int16_t)par;
        t.plo[lane] = nv.plo[a0 + lane]; t.phi[lane] = nv.phi[a0 + lane];
    }
    // depth by pointer jumping (root points at itself with depth 0)
    int dep = (lane > 0 && lane < m) ? 1 : 0;
    int anc = (lane > 0 && lane < m) ? par : 0;
#pragma unroll
    for (int r = 0; r < 5; r++) {
        const int da = __shfl_sync(0xffffffffu, dep, anc);
        const int aa = __shfl_sync(0xffffffffu, anc, anc);
        dep += da; anc = aa;
    }
    // children masks
    for (int v = 0; v < m; v++) {
        const uint32_t cm = __ballot_sync(0xffffffffu, lane > 0 && lane < m && par == v);
        if (lane == v) t.cmask[v] = cm;
    }
    int maxd = dep;
#pragma unroll
    for (int off = 16; off; off >>= 1) maxd = max(maxd, __shfl_xor_sync(0xffffffffu, maxd, off));
    if (lane < m) t.depth[lane] = (uint16_t)dep;
    __syncwarp();
    // all prefix gathers of the net up front
    for (int task = lane; task < 4 * (m - 1); task += 32) gather_task(g, t, task);
    __syncwarp();
    // bottom-up DP, deepest level first
    for (int d = maxd; d >= 1; d--) {
        uint32_t lv = __ballot_sync(0xffffffffu, lane < m && dep == d);
        while (lv) {
            const int v = __ffs(lv) - 1;
            lv &= lv - 1;
            span_table<false>(h, t, w, v, L);
            node_table(t, w, v, L);
            edge_table(h, t, w, v, L, nH, nV);
        }
    }
    span_table<false>(h, t, w, 0, L);
    const unsigned long long rk = root_min(t, w, L);
    if (lane == 0) t.span[0] = (uint8_t)(rk & 0xFF);
    __syncwarp();
    // top-down backtrack
    uint32_t seg = 0xFFFFFFFFu;
    for (int d = 1; d <= maxd; d++) {
        if (lane < m && dep == d) seg = backtrack_node(h, t, lane, L);
        __syncwarp();
    }
    if (lane < m) {
        if (o.rec_seg) o.rec_seg[o.rec_off[o.list_base + idx] + lane] = seg;
        else o.seg[a0 + lane] = seg;
    }
    if (lane == 0) {
        const uint32_t total = (uint32_t)(rk >> 8);
        if (o.rec_seg) o.rec_cost[o.list_base + idx] = total;
        else o.cost[net] = total;
    }
    if (commit && lane > 0 && lane < m) commit_edge(g, h, xx, yy, t.x[par], t.y[par], seg);
}

// CTA path: one 256-thread block per net with > 32 nodes.
__global__ void __launch_bounds__(FGR_CTA_THREADS) k_dp_large(GridView g, NetsView nv, const int32_t* __restrict__ list,
                                                               int count, Out o, int commit, int32_t* reset_ptr) {
    extern __shared__ __align__(16) unsigned char smem[];
    Hdr* h = reinterpret_cast<Hdr*>(smem);
    __shared__ int s_maxd;
    __shared__ unsigned long long s_root;
    init_hdr(h, g);
    if (threadIdx.x == 0) s_maxd = 0;
    if (reset_ptr && blockIdx.x == 0 && threadIdx.x == 0) *reset_ptr = 0;
    const int L = g.L, nH = g.h.cnt, nV = g.v.cnt;
    const int warp = threadIdx.x >> 5, lane = lane_id(), tid = threadIdx.x, T = blockDim.x;
    const int idx = blockIdx.x;
    const int net = list[idx];
    const int a0 = nv.off[net];
    const int m = nv.off[net + 1] - a0;
    unsigned char* base = smem + a16(sizeof(Hdr));
    WScr w = carve_wscr(base + (size_t)warp * wscr_bytes(L), L);
    Tabs t = carve_tabs(base + (size_t)FGR_WARPS_PER_CTA * wscr_bytes(L), m, L, nH, nV, true);
    for (int i = tid; i < m; i += T) {
        const int p = nv.par[a0 + i];
        t.x[i] = nv.x[a0 + i]; t.y[i] = nv.y[a0 + i]; t.par[i] = (int16_t)p;
        t.plo[i] = nv.plo[a0 + i]; t.phi[i] = nv.phi[a0 + i];
        t.depth[i] = i ? 1 : 0;
        t.anc[i] = (uint16_t)(i ? p : 0);
    }
    uint32_t* cnt = t.legH;   // child counts reuse the leg area before the gathers
    for (int i = tid; i <= m; i += T) cnt[i] = 0;
    __syncthreads();
    for (int i = 1 + tid; i < m; i += T) atomicAdd(&cnt[t.par[i]], 1u);
    // depth by pointer jumping: ceil(log2 m) rounds
    for (int r = 1; r < m; r <<= 1) {
        uint16_t nd[8], na[8];
#pragma unroll
        for (int q = 0; q < 8; q++) {
            const int i = tid + q * T;
            if (i < m) { const int an = t.anc[i]; nd[q] = t.depth[i] + t.depth[an]; na[q] = t.anc[an]; }
        }
        __syncthreads();
#pragma unroll
        for (int q = 0; q < 8; q++) {
            const int i = tid + q * T;
            if (i < m) { t.depth[i] = nd[q]; t.anc[i] = na[q]; }
        }
        __syncthreads();
    }
    // child CSR: exclusive scan of counts by warp 0
    if (warp == 0) {
        uint32_t carry = 0;
        for (int c0 = 0; c0 <= m; c0 += 32) {
            const int i = c0 + lane;
            const uint32_t v = i <= m ? cnt[i] : 0;
            uint32_t inc = v;
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                const uint32_t q = __shfl_up_sync(0xffffffffu, inc, off);
                if (lane >= off) inc += q;
            }
            if (i <= m) t.cstart[i] = (uint16_t)(carry + inc - v);
            carry += __shfl_sync(0xffffffffu, inc, 31);
        }
    }
    int md = 0;
    for (int i = tid; i < m; i += T) md = max(md, (int)t.depth[i]);
    atomicMax(&s_maxd, md);
    __syncthreads();
    for (int i = tid; i <= m; i += T) cnt[i] = t.cstart[i];
    __syncthreads();
    for (int i = 1 + tid; i < m; i += T) t.clist[atomicAdd(&cnt[t.par[i]], 1u)] = (uint16_t)i;
    __syncthreads();
    for (int task = tid; task < 4 * (m - 1); task += T) gather_task(g, t, task);
    __syncthreads();
    const int maxd = s_maxd;
    for (int d = maxd; d >= 1; d--) {
        for (int c0 = warp * 32; c0 < m; c0 += T) {
            const int i = c0 + lane;
            uint32_t lv = __ballot_sync(0xffffffffu, i < m && t.depth[i] == d);
            while (lv) {
                const int v = c0 + __ffs(lv) - 1;
                lv &= lv - 1;
                span_table<true>(h, t, w, v, L);
                node_table(t, w, v, L);
                edge_table(h, t, w, v, L, nH, nV);
            }
        }
        __syncthreads();
    }
    if (warp == 0) {
        span_table<true>(h, t, w, 0, L);
        const unsigned long long rk = root_min(t, w, L);
        if (lane == 0) { t.span[0] = (uint8_t)(rk & 0xFF); s_root = rk; }
    }
    __syncthreads();
    for (int d = 1; d <= maxd; d++) {
        for (int i = tid; i < m; i += T)
            if (t.depth[i] == d) {
                const uint32_t s = backtrack_node(h, t, i, L);
                if (o.rec_seg) o.rec_seg[o.rec_off[o.list_base + idx] + i] = s;
                else o.seg[a0 + i] = s;
                if (commit) {
                    const int u = t.par[i];
                    commit_edge(g, h, t.x[i], t.y[i], t.x[u], t.y[u], s);
                }
            }
        __syncthreads();
    }
    if (tid == 0) {
        const uint32_t total = (uint32_t)(s_root >> 8);
        if (o.rec_seg) { o.rec_seg[o.rec_off[o.list_base + idx]] = 0xFFFFFFFFu; o.rec_cost[o.list_base + idx] = total; }
        else { o.seg[a0] = 0xFFFFFFFFu; o.cost[net] = total; }
    }
}

// Commit from route records (multi-GPU: after the exchange every rank commits every net).
__global__ void __launch_bounds__(256) k_commit_records(GridView g, NetsView nv, const int32_t* __restrict__ list, int count,
                                                        const uint32_t* __restrict__ rec_seg,
                                                        const int32_t* __restrict__ rec_off, int list_base, int32_t* reset_ptr) {
    __shared__ Hdr hs;
    init_hdr(&hs, g);
    if (reset_ptr && blockIdx.x == 0 && threadIdx.x == 0) *reset_ptr = 0;
    __syncthreads();
    const int warp = (int)((blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5);
    const int nwarps = (int)((gridDim.x * (size_t)blockDim.x) >> 5);
    for (int idx = warp; idx < count; idx += nwarps) {
        const int net = list[idx];
        const int a0 = nv.off[net], m = nv.off[net + 1] - a0;
        const uint32_t* rs = rec_seg + rec_off[list_base + idx];
        for (int i = 1 + lane_id(); i < m; i += 32) {
            const int u = nv.par[a0 + i];
            commit_edge(g, &hs, nv.x[a0 + i], nv.y[a0 + i], nv.x[a0 + u], nv.y[a0 + u], rs[i]);
        }
    }
}

}  // namespace

size_t fgr_dp_smem_small(const fgr_grid* g) {
    return a16(sizeof(Hdr)) + (size_t)FGR_WARPS_PER_CTA * (tabs_bytes(32, g->L, g->nH, g->nV, false) + wscr_bytes(g->L));
}

size_t fgr_dp_smem_large(const fgr_grid* g, int m) {
    return a16(sizeof(Hdr)) + (size_t)FGR_WARPS_PER_CTA * wscr_bytes(g->L) + tabs_bytes(m, g->L, g->nH, g->nV, true);
}

cudaError_t fgr_launch_dp(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int count, int nlarge,
                          int maxm_large, uint32_t* seg_out, uint32_t* cost_out, uint32_t* rec_seg,
                          const int32_t* rec_off, uint32_t* rec_cost, int list_base, bool commit) {
    GridView v = g->view;
    v.seglist = g->d_list[g->parity];
    v.segcount = g->d_count + g->parity;
    // The other list was consumed by the refresh that ran before this launch: the
    // first kernel of this batch resets its length for the next commit.
    int32_t* reset = commit ? g->d_count + (g->parity ^ 1) : nullptr;
    Out o;
    o.seg = seg_out; o.cost = cost_out; o.rec_seg = rec_seg; o.rec_off = rec_off; o.rec_cost = rec_cost;
    o.list_base = list_base;
    cudaError_t e = cudaSuccess;
    static int configured = 0;
    if (!configured) {
        // opt in to the full shared memory minus each kernel's static shared memory
        cudaFuncAttributes fa;
        e = cudaFuncGetAttributes(&fa, k_dp_large);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(k_dp_large, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     g->max_smem - (int)fa.sharedSizeBytes);
        if (e == cudaSuccess) e = cudaFuncGetAttributes(&fa, k_dp_small);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(k_dp_small, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     g->max_smem - (int)fa.sharedSizeBytes);
        if (e != cudaSuccess) return e;
        configured = 1;
    }
    if (nlarge > 0) {
        k_dp_large<<<nlarge, FGR_CTA_THREADS, fgr_dp_smem_large(g, maxm_large), st>>>(v, nv, list, nlarge, o,
                                                                                       commit ? 1 : 0, reset);
        reset = nullptr;
        g->stats.kernel_launches++;
        e = cudaGetLastError();
        if (e != cudaSuccess) return e;
    }
    const int nsmall = count - nlarge;
    if (nsmall > 0) {
        Out os = o;
        os.list_base = list_base + nlarge;
        k_dp_small<<<(nsmall + FGR_WARPS_PER_CTA - 1) / FGR_WARPS_PER_CTA, FGR_CTA_THREADS, fgr_dp_smem_small(g), st>>>(
            v, nv, list + nlarge, nsmall, os, commit ? 1 : 0, reset);
        reset = nullptr;
        g->stats.kernel_launches++;
        e = cudaGetLastError();
        if (e != cudaSuccess) return e;
    }
    if (reset) return cudaMemsetAsync(reset, 0, sizeof(int32_t), st);
    return cudaSuccess;
}

cudaError_t fgr_launch_commit(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int count,
                              const uint32_t* rec_seg, const int32_t* rec_off, int list_base) {
    GridView v = g->view;
    v.seglist = g->d_list[g->parity];
    v.segcount = g->d_count + g->parity;
    int blocks = (count + 7) / 8;
    if (blocks > g->num_sms * 8) blocks = g->num_sms * 8;
    if (blocks < 1) blocks = 1;
    k_commit_records<<<blocks, 256, 0, st>>>(v, nv, list, count, rec_seg, rec_off, list_base,
                                             g->d_count + (g->parity ^ 1));
    g->stats.kernel_launches++;
    return cudaGetLastError();
}

void fgr_flip_lists(fgr_grid* g) { g->parity ^= 1; }
