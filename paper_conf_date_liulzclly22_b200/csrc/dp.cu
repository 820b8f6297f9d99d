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
// B200 mapping.  The layer count LT is a template parameter (every per-layer
// loop is unrolled exactly).  This file holds:
//   * k_dp_two: 2-node nets (half of all nets), one thread per net, the whole DP
//     in registers;
//   * k_dp_large: the round-1 kernel for nets of 65..~1.3k nodes, one 512-thread
//     CTA per net, heavy-path product form (the root path walked with transfer
//     matrices precomputed by helper warps, other paths by path walks) — selected
//     only by FGR_DP_HEAVY; the default large-net kernel is k_dp_tree (dp_tree.cu);
//   * k_commit_records: the S6 commit from exchanged route records (multi-GPU);
//   * launch_lt: the per-batch launcher (size classes on side streams, the
//     kernel of each large-net bucket by fgr_set_dp_policy, one grid-wide commit
//     of the tree-kernel nets after the join).
// All prefix gathers of a net are issued up front (costs are fixed during the
// DP); the per-node tables live in shared memory; each min-plus step is a DPX
// VIADDMNMX (sat_add).  Tie-breaks follow reading R11 exactly.
#include "dp_common.cuh"

namespace {

constexpr int kLargeWarps = 16;             // warps per CTA in k_dp_large (one path-walking group each)
constexpr int kFlowMax = 64;                // largest net of the dataflow kernel by default



struct Tabs {
    uint32_t* E;      // [m][LT]      E_v(lt) = c*(v -> parent, lt)
    uint32_t* legH;   // [m][2][nH]   0: row y_v, 1: row y_u   (x_v..x_u)
    uint32_t* legV;   // [m][2][nV]   0: col x_v, 1: col x_u   (y_v..y_u)
    uint32_t* aux;    // [m]  group path: children bitmask, then pointer-jumping ancestor
    int16_t* x;
    int16_t* y;
    int16_t* par;
    uint16_t* depth;
    uint16_t* cstart; // CTA path: child CSR [m+1]
    uint16_t* clist;  // CTA path: [m]
    uint16_t* anc;    // CTA path: pointer-jumping scratch [m], then the nodes sorted by level
    uint16_t* lvstart;// CTA path: level CSR [m+1]
    uint16_t* hv;     // CTA path: heavy child (0xFFFF = leaf)
    uint16_t* top;    // CTA path: top node of the heavy path holding v
    uint16_t* bot;    // CTA path: bottom (leaf) of the path topped by v
    uint16_t* pq;     // CTA path: path tops, deepest top first
    uint16_t* rpos;   // CTA path: index along the root path from its bottom (0xFFFF off the root path)
    uint16_t* rp;     // CTA path: root path nodes, bottom first
    uint16_t* argq;   // CTA path: root-path items whose recB/recE a helper fills in
    uint8_t* done;    // CTA path: E_v final (values pass)
    uint8_t* sready;  // CTA path: span_v final (backtrack)
    int8_t* plo;
    int8_t* phi;
    uint8_t* span;    // chosen via span (lo << 4) | hi  (low byte of the packed (value, lo, hi) key)
    uint8_t* recE;    // [m][LT] argmin ls of E_v(lt)
    uint8_t* recB;    // [m][LT] argmin span of B_v(ls)
};

struct WScr {          // per-group scratch
    unsigned long long* R;  // [LT][LT]  R(lo,b) = min_{hi >= b} key(lo,hi), key = F<<8 | lo<<4 | hi
    uint32_t* B;            // [LT]
};

__host__ __device__ inline size_t tabs_bytes(int m, int L, int nH, int nV, bool cta) {
    size_t b = 0;
    b += a16((size_t)m * L * 4);
    b += a16((size_t)m * 2 * nH * 4);
    b += a16((size_t)m * 2 * nV * 4);
    if (!cta) b += a16((size_t)m * 4);
    b += 4 * a16((size_t)m * 2);
    if (cta) b += 2 * a16((size_t)(m + 1) * 2) + 9 * a16((size_t)m * 2) + 2 * a16((size_t)m);
    b += 3 * a16((size_t)m);
    b += 2 * a16((size_t)m * L);
    return b;
}

__host__ __device__ inline size_t wscr_bytes(int L) { return a16((size_t)L * L * 8) + a16((size_t)L * 4); }

__device__ inline Tabs carve_tabs(unsigned char* p, int m, int L, int nH, int nV, bool cta) {
    Tabs t;
    t.E = (uint32_t*)p; p += a16((size_t)m * L * 4);
    t.legH = (uint32_t*)p; p += a16((size_t)m * 2 * nH * 4);
    t.legV = (uint32_t*)p; p += a16((size_t)m * 2 * nV * 4);
    t.aux = nullptr;
    if (!cta) { t.aux = (uint32_t*)p; p += a16((size_t)m * 4); }
    t.x = (int16_t*)p; p += a16((size_t)m * 2);
    t.y = (int16_t*)p; p += a16((size_t)m * 2);
    t.par = (int16_t*)p; p += a16((size_t)m * 2);
    t.depth = (uint16_t*)p; p += a16((size_t)m * 2);
    t.cstart = t.clist = t.anc = t.lvstart = t.hv = t.top = t.bot = t.pq = t.rpos = t.rp = t.argq = nullptr;
    t.done = t.sready = nullptr;
    if (cta) {
        t.cstart = (uint16_t*)p; p += a16((size_t)(m + 1) * 2);
        t.lvstart = (uint16_t*)p; p += a16((size_t)(m + 1) * 2);
        t.clist = (uint16_t*)p; p += a16((size_t)m * 2);
        t.anc = (uint16_t*)p; p += a16((size_t)m * 2);
        t.hv = (uint16_t*)p; p += a16((size_t)m * 2);
        t.top = (uint16_t*)p; p += a16((size_t)m * 2);
        t.bot = (uint16_t*)p; p += a16((size_t)m * 2);
        t.pq = (uint16_t*)p; p += a16((size_t)m * 2);
        t.rpos = (uint16_t*)p; p += a16((size_t)m * 2);
        t.rp = (uint16_t*)p; p += a16((size_t)m * 2);
        t.argq = (uint16_t*)p; p += a16((size_t)m * 2);
        t.done = (uint8_t*)p; p += a16((size_t)m);
        t.sready = (uint8_t*)p; p += a16((size_t)m);
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
    w.R = (unsigned long long*)p;
    w.B = (uint32_t*)(p + a16((size_t)L * L * 8));
    return w;
}



// Per-lane constants of the group lane that owns layer `gl` (= lo in the K rows, = lt in the edge step).
template <int LT>
struct LaneConst {
    uint32_t vme[LT];      // V(min(l, gl), max(l, gl)): via stack between layer l and this lane's layer
    uint32_t vp[LT];       // viapre[l]       (indexed only by compile-time l)
    uint32_t zl[LT];       // zlo[l]
    uint32_t hmask;        // layers with dir == H
    int my_dir, my_slot;
    __device__ __forceinline__ void load(const Hdr* h, int gl) {
        const int me = gl < LT ? gl : 0;
        const uint32_t vpm = h->viapre[me];
#pragma unroll
        for (int i = 0; i < LT; i++) {
            const uint32_t vi = h->viapre[i];
            vp[i] = vi;
            zl[i] = h->zlo[i];
            vme[i] = vi >= vpm ? vi - vpm : vpm - vi;   // viapre is non-decreasing
        }
        hmask = 0;
#pragma unroll
        for (int i = 0; i < LT; i++) hmask |= (h->dir[i] == 0 ? 1u : 0u) << i;
        my_dir = h->dir[me];
        my_slot = h->slot[me];
    }
};


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

// ------------------------------------------------------------- DP steps (one group of LT lanes)

// Packed G entry of a node without light children (K = V): value V(a,b), span (zlo[a], b).
__device__ __forceinline__ unsigned long long gclosed(const Hdr* h, int a, int b) {
    return ((unsigned long long)(h->viapre[b] - h->viapre[a]) << 8) | (unsigned)(h->zlo[a] << 4) | (unsigned)b;
}

// min of N packed keys as a balanced tree (dependency depth log2 N instead of N)
template <int N>
__device__ __forceinline__ unsigned long long tree_min(unsigned long long (&k)[N]) {
#pragma unroll
    for (int s = 1; s < N; s <<= 1)
#pragma unroll
        for (int i = 0; i + s < N; i += 2 * s) k[i] = k[i + s] < k[i] ? k[i + s] : k[i];
    return k[0];
}

// ------------------------------------------------------------- CTA kernel (nets > 32 nodes)
// Heavy-path form of the same recurrences.  Split the tree into heavy paths (heavy
// child = largest subtree).  With every child of v known except the heavy child h,
// Eq. (2) becomes a min-plus product in E_h:
//     B_v(ls) = min_l [ E_h(l) + G_v(min(l, a), max(l, b)) ],  a = min(ls, pin_lo), b = max(ls, pin_hi)
// where K_v(S) = V(S) + sum_{light c} min_{l in S} E_c(l) and G_v(a, b) = min over spans
// S = [lo, hi] with lo <= a, hi >= b of K_v(S).  Carrying packed (value, lo, hi) keys
// through G and through the min over l reproduces R11's lexicographic span choice
// exactly (the optimal span is S*_l of some optimal l).  Without light
// children K = V and G has a closed form.  A path is then walked bottom-up by one
// lane group with one short vector step per node, and paths run as a dataflow (a
// node waits only for its light children), so the CTA never synchronises per
// tree level.  The backtrack walks the same paths top-down.

// Demand-independent tree analysis of a large net in shared memory: depths, child CSR,
// level CSR, path decomposition (heavy child, path tops / bottoms) and the path queue.
__device__ __forceinline__ void large_prologue(const Tabs& t, const NetsView& nv, int a0, int m, int tid, int T,
                                               int warp, int lane, int* s_maxd, int* s_npaths, int* s_deep) {
    for (int i = tid; i < m; i += T) {
        const int p = nv.par[a0 + i];
        t.x[i] = nv.x[a0 + i]; t.y[i] = nv.y[a0 + i]; t.par[i] = (int16_t)p;
        t.plo[i] = nv.plo[a0 + i]; t.phi[i] = nv.phi[a0 + i];
        t.depth[i] = i ? 1 : 0;
        t.anc[i] = (uint16_t)(i ? p : 0);
        t.done[i] = 0; t.sready[i] = 0;
    }
    uint32_t* cnt = t.legH;   // scratch in the leg areas before the gathers
    uint32_t* dcnt = t.legV;
    for (int i = tid; i <= m; i += T) { cnt[i] = 0; dcnt[i] = 0; }
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
    int md = 0;
    for (int i = tid; i < m; i += T) {
        md = max(md, (int)t.depth[i]);
        atomicAdd(&dcnt[t.depth[i]], 1u);
    }
    atomicMax(&(*s_maxd), md);
    __syncthreads();
    const int maxd = (*s_maxd);
    // warp 0: child CSR; warp 1: level CSR (exclusive scans)
    if (warp < 2) {
        const uint32_t* src = warp == 0 ? cnt : dcnt;
        uint16_t* dst = warp == 0 ? t.cstart : t.lvstart;
        const int n = warp == 0 ? m : maxd + 1;
        uint32_t carry = 0;
        for (int c0 = 0; c0 <= n; c0 += 32) {
            const int i = c0 + lane;
            const uint32_t v = i <= n ? src[i] : 0;
            uint32_t inc = v;
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                const uint32_t q = __shfl_up_sync(0xffffffffu, inc, off);
                if (lane >= off) inc += q;
            }
            if (i <= n) dst[i] = (uint16_t)(carry + inc - v);
            carry += __shfl_sync(0xffffffffu, inc, 31);
        }
    }
    __syncthreads();
    for (int i = tid; i <= m; i += T) cnt[i] = t.cstart[i];
    for (int i = tid; i <= maxd; i += T) dcnt[i] = t.lvstart[i];
    __syncthreads();
    for (int i = tid; i < m; i += T) {
        if (i > 0) t.clist[atomicAdd(&cnt[t.par[i]], 1u)] = (uint16_t)i;
        t.anc[atomicAdd(&dcnt[t.depth[i]], 1u)] = (uint16_t)i;   // nodes grouped by level, shallow first
    }
    __syncthreads();
    // Path decomposition: the ancestors of the deepest node (ties: smallest index)
    // form the root path, every other node continues through its smallest-index
    // child.  Any decomposition is exact; this one puts the deepest chain on one path.
    if (tid == 0) (*s_deep) = 0x7FFFFFFF;
    __syncthreads();
    for (int v = tid; v < m; v += T)
        if (t.depth[v] == maxd) atomicMin(&(*s_deep), v);
    for (int v = tid; v < m; v += T) {
        int best = -1;
        for (int k = t.cstart[v]; k < t.cstart[v + 1]; k++) {
            const int ch = t.clist[k];
            if (best < 0 || ch < best) best = ch;
        }
        t.hv[v] = best < 0 ? (uint16_t)0xFFFF : (uint16_t)best;
    }
    __syncthreads();
    if (tid == 0)
        for (int w = (*s_deep); w > 0; w = t.par[w]) t.hv[t.par[w]] = (uint16_t)w;
    __syncthreads();
    // top of each node's heavy path by pointer jumping over heavy edges
    for (int v = tid; v < m; v += T) t.top[v] = (v > 0 && t.hv[t.par[v]] == v) ? (uint16_t)t.par[v] : (uint16_t)v;
    __syncthreads();
    for (int r = 1; r <= maxd; r <<= 1) {
        uint16_t nt[8];
#pragma unroll
        for (int q = 0; q < 8; q++) {
            const int i = tid + q * T;
            if (i < m) nt[q] = t.top[t.top[i]];
        }
        __syncthreads();
#pragma unroll
        for (int q = 0; q < 8; q++) {
            const int i = tid + q * T;
            if (i < m) t.top[i] = nt[q];
        }
        __syncthreads();
    }
    for (int v = tid; v < m; v += T)
        if (t.hv[v] == 0xFFFF) t.bot[t.top[v]] = (uint16_t)v;
    __syncthreads();
    for (int v = tid; v < m; v += T)
        t.rpos[v] = t.top[v] == 0 ? (uint16_t)(t.depth[t.bot[0]] - t.depth[v]) : (uint16_t)0xFFFF;
    // path tops, deepest first (a light child's top is deeper than its parent's path top)
    if (warp == 0) {
        int n = 0;
        for (int c0 = m - 1; c0 >= 0; c0 -= 32) {
            const int k = c0 - lane;
            const int v = k >= 0 ? t.anc[k] : 0;
            const bool is_top = k >= 0 && t.top[v] == v;
            const unsigned b = __ballot_sync(0xffffffffu, is_top);
            if (is_top) t.pq[n + __popc(b & ((1u << lane) - 1u))] = (uint16_t)v;
            n += __popc(b);
        }
        if (lane == 0) (*s_npaths) = n;
    }
}

__device__ __forceinline__ int ld_flag(const uint8_t* f) { return *(volatile const uint8_t*)f; }

constexpr int kMR = 16;   // matrix ring slots (root-path transfer matrices in flight)
template <int LT> struct MStride { static constexpr int v = (LT + 3) & ~3; };

// Wait for v's light children (all children but the heavy one), then build the packed
// dominance table G_v of K_v in the warp's scratch w.R (lane = lo rows, then lane = b columns).
template <int LT>
__device__ __forceinline__ void build_G(const LaneConst<LT>& c, const Tabs& t, const WScr& w, int v, int gl,
                                        unsigned gmask) {
    const int hvv = t.hv[v];
    const int k0 = t.cstart[v], k1 = t.cstart[v + 1];
    for (int k = k0 + gl; k < k1; k += LT) {
        const int ch = t.clist[k];
        if (ch != hvv) {
            int spins = 0;
            while (ld_flag(&t.done[ch]) == 0)
                if (++spins > 64) __nanosleep(20);   // short busy phase first: this may be the critical walker
        }
    }
    __syncwarp(gmask);
    __threadfence_block();
    const int lo = gl;
    uint32_t acc[LT];
#pragma unroll
    for (int hi = 0; hi < LT; hi++) acc[hi] = hi >= lo ? c.vme[hi] : FGR_INF;
    for (int k = k0; k < k1; k++) {
        const int ch = t.clist[k];
        if (ch == hvv) continue;
        const uint32_t* Ec = t.E + (size_t)ch * LT;
        uint32_t run = FGR_INF;
#pragma unroll
        for (int hi = 0; hi < LT; hi++) {
            const uint32_t e = Ec[hi];
            if (hi >= lo) { run = min(run, e); acc[hi] = sat_add(acc[hi], run); }
        }
    }
    unsigned long long run = ~0ull;
#pragma unroll
    for (int hi = LT - 1; hi >= 0; hi--)
        if (hi >= lo) {
            const unsigned long long key = ((unsigned long long)acc[hi] << 8) | (unsigned)(lo << 4) | (unsigned)hi;
            run = key < run ? key : run;
            w.R[lo * LT + hi] = run;
        }
    __syncwarp(gmask);
    const int bcol = gl;
    unsigned long long pr = ~0ull;
#pragma unroll
    for (int a = 0; a < LT; a++)
        if (a <= bcol) {
            const unsigned long long x = w.R[a * LT + bcol];
            pr = x < pr ? x : pr;
            w.R[a * LT + bcol] = pr;
        }
    __syncwarp(gmask);
}

// One non-root node of a path walk in product form (G_v already built when light):
// B_v / recB_v from E_h (lanes of Eprev), then E_v / recE_v.  Returns this lane's E_v.
template <int LT>
__device__ __forceinline__ uint32_t path_node(const LaneConst<LT>& c, const Tabs& t, const WScr& w, int v, uint32_t Eprev,
                                              bool has_prev, bool light, int gl, int gbase, unsigned gmask, int nH,
                                              int nV, uint32_t opp, bool store_E, const uint32_t* hm) {
    const int plo = t.plo[v], phi = t.phi[v];
    const int ls = gl;
    int a0 = ls, b0 = ls;
    if (plo >= 0) { a0 = min(a0, plo); b0 = max(b0, phi); }
    unsigned long long bk;
    if (light) {
        if (!has_prev) bk = w.R[a0 * LT + b0];
        else {
            unsigned long long gk[LT];
#pragma unroll
            for (int l = 0; l < LT; l++) gk[l] = w.R[min(a0, l) * LT + max(b0, l)];
#pragma unroll
            for (int l = 0; l < LT; l++) {
                const uint32_t e = __shfl_sync(gmask, Eprev, gbase + l);
                gk[l] = ((unsigned long long)sat_add(e, (uint32_t)(gk[l] >> 8)) << 8) | (gk[l] & 0xFFull);
            }
            bk = tree_min<LT>(gk);
        }
    } else {
        uint32_t va0 = 0, vb0 = 0, za0 = 0;
#pragma unroll
        for (int l = 0; l < LT; l++) {
            va0 = (l == a0) ? c.vp[l] : va0;
            vb0 = (l == b0) ? c.vp[l] : vb0;
            za0 = (l == a0) ? c.zl[l] : za0;
        }
        if (!has_prev) bk = ((unsigned long long)(vb0 - va0) << 8) | (za0 << 4) | (unsigned)b0;
        else {
            unsigned long long kk[LT];
#pragma unroll
            for (int l = 0; l < LT; l++) {
                const uint32_t e = __shfl_sync(gmask, Eprev, gbase + l);
                const bool la = l < a0, lb = l > b0;
                const uint32_t va = la ? c.vp[l] : va0, vb = lb ? c.vp[l] : vb0;
                const uint32_t za = la ? c.zl[l] : za0;
                const uint32_t bb = lb ? (uint32_t)l : (uint32_t)b0;
                kk[l] = ((unsigned long long)sat_add(e, vb - va) << 8) | (za << 4) | bb;
            }
            bk = tree_min<LT>(kk);
        }
    }
    const uint32_t Bv = (uint32_t)(bk >> 8);
    t.recB[(size_t)v * LT + ls] = (uint8_t)(bk & 0xFF);
    const int lt = gl;
    const int u = t.par[v];
    const int xv = t.x[v], yv = t.y[v], xu = t.x[u], yu = t.y[u];
    uint32_t best = FGR_INF;
    int bls = lt;
    uint32_t Bl[LT];
#pragma unroll
    for (int l = 0; l < LT; l++) Bl[l] = __shfl_sync(gmask, Bv, gbase + l);
    if (hm) {                                     // hybrid edge: min-plus with the precomputed M_e
#pragma unroll
        for (int l = 0; l < LT; l++) {
            const uint32_t cst = sat_add(Bl[l], hm[l]);
            if (cst < best) { best = cst; bls = l; }
        }
    } else if (yv == yu || xv == xu) {
        const int de = (yv == yu) ? 0 : 1;
        if (c.my_dir == de) {
            const uint32_t leg = de == 0 ? t.legH[(size_t)v * 2 * nH + c.my_slot] : t.legV[(size_t)v * 2 * nV + c.my_slot];
            best = sat_add(Bv, leg);
        }
    } else {
        const bool b0v = c.my_dir == 1;
        const uint32_t leg2 = b0v ? t.legV[((size_t)v * 2 + 1) * nV + c.my_slot] : t.legH[((size_t)v * 2 + 1) * nH + c.my_slot];
        const uint32_t* l1 = b0v ? t.legH + (size_t)v * 2 * nH : t.legV + (size_t)v * 2 * nV;
        int sidx = 0;
#pragma unroll
        for (int l = 0; l < LT; l++)
            if ((opp >> l) & 1u) {
                const uint32_t cst = sat_add(sat_add(sat_add(Bl[l], l1[sidx]), c.vme[l]), leg2);
                if (cst < best) { best = cst; bls = l; }
                sidx++;
            }
    }
    if (store_E) t.E[(size_t)v * LT + lt] = best;
    t.recE[(size_t)v * LT + lt] = (uint8_t)bls;
    return best;
}

// Transfer matrix of node v (values only): E_v(lt) = min_l [E_h(l) + M_v(l, lt)],
// M_v(l, lt) = min_ls [C_v(l, ls) + W_v(ls, lt)], C_v(l, ls) = value of G_v(hull(l, ls, pins)).
// Exact: min-plus distributes over the saturating sums.  Lane lt writes column lt.
template <int LT>
__device__ __forceinline__ void build_M(const Hdr* h, const LaneConst<LT>& c, const Tabs& t, const WScr& w, int v,
                                        bool light, int gl, int nH, int nV, uint32_t opp, uint32_t* col,
                                        const uint32_t* hm) {
    const int plo = t.plo[v], phi = t.phi[v];
    const int lt = gl;
    const int u = t.par[v];
    const int xv = t.x[v], yv = t.y[v], xu = t.x[u], yu = t.y[u];
    const bool straight = (yv == yu) || (xv == xu);
    uint32_t legS = FGR_INF, leg2 = 0;
    const uint32_t* l1 = nullptr;
    if (straight) {
        const int de = (yv == yu) ? 0 : 1;
        if (c.my_dir == de) legS = de == 0 ? t.legH[(size_t)v * 2 * nH + c.my_slot] : t.legV[(size_t)v * 2 * nV + c.my_slot];
    } else {
        const bool b0v = c.my_dir == 1;
        leg2 = b0v ? t.legV[((size_t)v * 2 + 1) * nV + c.my_slot] : t.legH[((size_t)v * 2 + 1) * nH + c.my_slot];
        l1 = b0v ? t.legH + (size_t)v * 2 * nH : t.legV + (size_t)v * 2 * nV;
    }
    for (int l = 0; l < LT; l++) {
        uint32_t best = FGR_INF;
        if (hm) {   // hybrid edge: W_v(ls, lt) = M_e(ls, lt)
#pragma unroll
            for (int ls = 0; ls < LT; ls++) {
                int a = ls, b = ls;
                if (plo >= 0) { a = min(a, plo); b = max(b, phi); }
                a = min(a, l); b = max(b, l);
                const uint32_t cv = light ? (uint32_t)(w.R[a * LT + b] >> 8) : h->viapre[b] - h->viapre[a];
                best = min(best, sat_add(cv, hm[ls]));
            }
        } else if (straight) {
            if (legS != FGR_INF) {
                int a = lt, b = lt;
                if (plo >= 0) { a = min(a, plo); b = max(b, phi); }
                a = min(a, l); b = max(b, l);
                const uint32_t cv = light ? (uint32_t)(w.R[a * LT + b] >> 8) : h->viapre[b] - h->viapre[a];
                best = sat_add(cv, legS);
            }
        } else {
            int sidx = 0;
#pragma unroll
            for (int ls = 0; ls < LT; ls++)
                if ((opp >> ls) & 1u) {
                    int a = ls, b = ls;
                    if (plo >= 0) { a = min(a, plo); b = max(b, phi); }
                    a = min(a, l); b = max(b, l);
                    const uint32_t cv = light ? (uint32_t)(w.R[a * LT + b] >> 8) : h->viapre[b] - h->viapre[a];
                    const uint32_t cst = sat_add(sat_add(sat_add(cv, l1[sidx]), c.vme[ls]), leg2);
                    best = min(best, cst);
                    sidx++;
                }
        }
        col[lt * MStride<LT>::v + l] = best;
    }
}

#ifdef FGR_TIMING
#define TMARK(i) do { if (threadIdx.x == 0) tm[i] = clock64(); } while (0)
#else
#define TMARK(i) do { } while (0)
#endif



template <int LT>
__global__ void __launch_bounds__(32 * kLargeWarps, 1) k_dp_large(GridView g, NetsView nv, const int32_t* __restrict__ list,
                                                                  int count, Out o, int commit, Prep prep,
                                                                  HybView hy) {
    constexpr int G = 1;   // one lane group per warp: a path walk never shares its warp's issue slots
    extern __shared__ __align__(16) unsigned char smem[];
    Hdr* h = reinterpret_cast<Hdr*>(smem);
    __shared__ int s_maxd, s_ticket, s_ticket2, s_npaths, s_deep;
    __shared__ unsigned long long s_root;
    init_hdr(h, g);
    if (threadIdx.x == 0) { s_maxd = 0; s_root = ~0ull; s_ticket = 0; s_ticket2 = 0; s_npaths = 0; }
    const int nH = g.h.cnt, nV = g.v.cnt;
    const int warp = threadIdx.x >> 5, lane = lane_id(), tid = threadIdx.x, T = blockDim.x;
    const int gi = lane / LT < G ? lane / LT : G;
    const int gl = lane - gi * LT;
    const bool glane = gi < G && gl < LT;
    const int gbase = gi * LT;
    const unsigned gmask = glane ? (((1u << LT) - 1u) << gbase) : 0u;
    const int idx = blockIdx.x;
#ifdef FGR_TIMING
    long long tm[8];
#endif
    TMARK(0);
    const int net = list[idx];
    const int a0 = nv.off[net];
    const int m = nv.off[net + 1] - a0;
    const int hnet = hy.net ? hy.net[net] : -1;
    // hybrid edge of node v: its transfer matrix column for lt = gl (nullptr for an L edge)
    auto hmat = [&](int v) -> const uint32_t* {
        if (hnet < 0) return nullptr;
        const int hs = hy.slot[a0 + v];
        return hs >= 0 ? hy.M + ((size_t)hs * LT + gl) * LT : nullptr;
    };
    unsigned char* base = smem + a16(sizeof(Hdr));
    const WScr w = carve_wscr(base + ((size_t)warp * G + (gi < G ? gi : 0)) * wscr_bytes(LT), LT);
    const Tabs t = carve_tabs(base + (size_t)kLargeWarps * G * wscr_bytes(LT), m, LT, nH, nV, true);
    if (prep.cs) {
        // tree analysis precomputed once per stage by k_large_prep: just load it
        for (int i = tid; i < m; i += T) {
            t.x[i] = nv.x[a0 + i]; t.y[i] = nv.y[a0 + i]; t.par[i] = (int16_t)nv.par[a0 + i];
            t.plo[i] = nv.plo[a0 + i]; t.phi[i] = nv.phi[a0 + i];
            t.cstart[i] = prep.cs[a0 + i]; t.clist[i] = prep.cl[a0 + i]; t.hv[i] = prep.hv[a0 + i];
            t.bot[i] = prep.bot[a0 + i]; t.pq[i] = prep.pq[a0 + i]; t.rpos[i] = prep.rpos[a0 + i];
            t.done[i] = 0; t.sready[i] = 0;
        }
        if (tid == 0) { t.cstart[m] = (uint16_t)(m - 1); s_npaths = prep.npaths[net]; }
        __syncthreads();
    } else {
        large_prologue(t, nv, a0, m, tid, T, warp, lane, &s_maxd, &s_npaths, &s_deep);
    }
    LaneConst<LT> c;
    c.load(h, gl);
    TMARK(1);
    pdl_wait();   // everything above is demand-independent; the refresh must be done before the gathers
#pragma unroll 2
    for (int task = tid; task < 4 * (m - 1); task += T) gather_task(g, t, task);
    __syncthreads();
    TMARK(2);
    const int npaths = s_npaths;
    // ---------------- values: bottom-up path walks
    // warp 0 walks the root path; the other warps walk the remaining paths (deepest tops
    // first), then precompute root-path transfer matrices ahead of warp 0 and fill in the
    // recB/recE of the nodes warp 0 passed with a matrix step.
    __shared__ int s_K, s_mnext, s_anext, s_acount, s_wdone;
    __shared__ int sstate[kMR];   // slot state: generation * 4 + {0 free, 1 writing, 2 ready}
    uint32_t* mslots = reinterpret_cast<uint32_t*>(base + (size_t)kLargeWarps * G * wscr_bytes(LT) +
                                                   tabs_bytes(m, LT, nH, nV, true));
    for (int v = tid; v < m; v += T)
        if (t.rpos[v] != 0xFFFF) t.rp[t.rpos[v]] = (uint16_t)v;
    if (tid == 0) { s_K = t.rpos[0] + 1; s_mnext = 1; s_anext = 0; s_acount = 0; s_wdone = 0; }
    if (tid < kMR) sstate[tid] = (tid == 0 ? kMR : tid) * 4;
    __syncthreads();
    const int K = s_K;
    if (glane) {
        const uint32_t opp = c.my_dir == 1 ? c.hmask : (~c.hmask & ((1u << LT) - 1u));   // bend partner layers
        if (warp == 0) {
            // ---- root-path walker
            uint32_t Eprev = FGR_INF;
#ifdef FGR_TIMING
            long long w_slot = 0, w_inline = 0, w_fast = 0, w_x;
#endif
            for (int k = 0; k < K; k++) {
                const int v = t.rp[k];
                if (v == 0) {
                    // generalised Eq. (4): min over l of E_h(l) + G(hull({l} + pins)) (any span for a Steiner root)
                    const bool light = (t.cstart[1] - t.cstart[0]) > 1;
                    if (light) build_G<LT>(c, t, w, 0, gl, gmask);
                    const int plo = t.plo[0], phi = t.phi[0];
                    const int ra = plo >= 0 ? plo : LT - 1, rb = plo >= 0 ? phi : 0;
                    unsigned long long kk[LT];
#pragma unroll
                    for (int l = 0; l < LT; l++) {
                        const uint32_t e = __shfl_sync(gmask, Eprev, gbase + l);
                        const int a = min(ra, l), b = max(rb, l);
                        const unsigned long long gk = light ? w.R[a * LT + b] : gclosed(h, a, b);
                        kk[l] = ((unsigned long long)sat_add(e, (uint32_t)(gk >> 8)) << 8) | (gk & 0xFFull);
                    }
                    const unsigned long long best = tree_min<LT>(kk);
                    if (gl == 0) { s_root = best; t.span[0] = (uint8_t)(best & 0xFF); }
                    __syncwarp(gmask);
                    __threadfence_block();
                    if (gl == 0) { t.done[0] = 1; *(volatile uint8_t*)&t.sready[0] = 1; }
                    break;
                }
                bool fast = false;
#ifdef FGR_TIMING
                w_x = clock64();
#endif
                if (k > 0) {
                    const int sl = k % kMR;
                    for (;;) {
                        const int st = *(volatile int*)&sstate[sl];
                        if (st == k * 4 + 2) { fast = true; break; }
                        if (st == k * 4) {
                            int old = 0;
                            if (gl == 0) old = atomicCAS(&sstate[sl], k * 4, (k + kMR) * 4);   // not ready: go inline
                            old = __shfl_sync(gmask, old, gbase);
                            if (old == k * 4) break;
                            continue;
                        }
                        // a helper is writing this matrix: busy-wait (a sleeping walker oversleeps)
                    }
#ifdef FGR_TIMING
                    w_slot += clock64() - w_x; w_x = clock64();
#endif
                    if (fast) {
                        __threadfence_block();
                        const uint32_t* col = mslots + (size_t)sl * LT * MStride<LT>::v + gl * MStride<LT>::v;
                        unsigned long long dummy;
                        (void)dummy;
                        uint32_t ev[LT];
#pragma unroll
                        for (int l = 0; l < LT; l++) ev[l] = sat_add(__shfl_sync(gmask, Eprev, gbase + l), col[l]);
#pragma unroll
                        for (int s2 = 1; s2 < LT; s2 <<= 1)
#pragma unroll
                            for (int i = 0; i + s2 < LT; i += 2 * s2) ev[i] = min(ev[i], ev[i + s2]);
                        const uint32_t Ev = ev[0];
                        t.E[(size_t)v * LT + gl] = Ev;
                        __syncwarp(gmask);
                        if (gl == 0) {
                            *(volatile int*)&sstate[sl] = (k + kMR) * 4;   // slot free for item k + kMR
                            t.argq[s_acount] = (uint16_t)k;
                            __threadfence_block();
                            *(volatile int*)&s_acount = s_acount + 1;
                        }
                        Eprev = Ev;
#ifdef FGR_TIMING
                        w_fast += clock64() - w_x;
#endif
                        continue;
                    }
                }
                const bool light = (t.cstart[v + 1] - t.cstart[v]) > 1;
                if (light) build_G<LT>(c, t, w, v, gl, gmask);
                Eprev = path_node<LT>(c, t, w, v, Eprev, k > 0, light, gl, gbase, gmask, nH, nV, opp, true, hmat(v));
                __syncwarp(gmask);
                __threadfence_block();
#ifdef FGR_TIMING
                w_inline += clock64() - w_x;
#endif
            }
            if (gl == 0) *(volatile int*)&s_wdone = 1;
#ifdef FGR_TIMING
            if (gl == 0 && m > 880) printf("WALK m=%d K=%d fast=%d t=%lld slot=%lld inline=%lld fastc=%lld\n", m, K, s_acount,
                                           clock64() - tm[2], w_slot, w_inline, w_fast);
#endif
        } else {
            // ---- the other paths, deepest tops first (pq[npaths-1] is the root path)
            for (;;) {
                int p = 0;
                if (gl == 0) p = atomicAdd(&s_ticket, 1);
                p = __shfl_sync(gmask, p, gbase);
                if (p >= npaths - 1) break;
                const int tp = t.pq[p];
                int v = t.bot[tp];
                uint32_t Eprev = FGR_INF;
                bool has_prev = false;
                for (;;) {
                    const bool light = (t.cstart[v + 1] - t.cstart[v]) > 1;
                    if (light) build_G<LT>(c, t, w, v, gl, gmask);
                    const uint32_t Ev = path_node<LT>(c, t, w, v, Eprev, has_prev, light, gl, gbase, gmask, nH, nV, opp, true,
                                                      hmat(v));
                    if (v == tp) {   // only path tops are read by other warps (as light children)
                        __syncwarp(gmask);
                        __threadfence_block();
                        if (gl == 0) *(volatile uint8_t*)&t.done[v] = 1;
                        break;
                    }
                    Eprev = Ev;
                    has_prev = true;
                    v = t.par[v];
                }
            }
            // ---- root-path transfer matrices ahead of the walker
            for (;;) {
                int k = 0;
                if (gl == 0) k = atomicAdd(&s_mnext, 1);
                k = __shfl_sync(gmask, k, gbase);
                if (k >= K - 1) break;
                const int sl = k % kMR;
                int st;
                for (;;) {
                    st = *(volatile int*)&sstate[sl];
                    if ((st >> 2) >= k) break;
                    __nanosleep(32);
                }
                if (st != k * 4) continue;   // the walker passed this item already
                const int v = t.rp[k];
                const bool light = (t.cstart[v + 1] - t.cstart[v]) > 1;
                if (light) build_G<LT>(c, t, w, v, gl, gmask);   // waits for v's light children
                int old = 0;
                if (gl == 0) old = atomicCAS(&sstate[sl], k * 4, k * 4 + 1);
                old = __shfl_sync(gmask, old, gbase);
                if (old != k * 4) continue;
                build_M<LT>(h, c, t, w, v, light, gl, nH, nV, opp, mslots + (size_t)sl * LT * MStride<LT>::v, hmat(v));
                __syncwarp(gmask);
                __threadfence_block();
                if (gl == 0) *(volatile int*)&sstate[sl] = k * 4 + 2;
            }
            // ---- recB / recE of the root-path nodes the walker passed with a matrix step
            for (;;) {
                int j = 0;
                if (gl == 0) j = atomicAdd(&s_anext, 1);
                j = __shfl_sync(gmask, j, gbase);
                int cnt;
                bool over = false;
                for (;;) {
                    cnt = *(volatile int*)&s_acount;
                    if (j < cnt) break;
                    if (*(volatile int*)&s_wdone) {
                        cnt = *(volatile int*)&s_acount;
                        if (j >= cnt) over = true;
                        break;
                    }
                    __nanosleep(64);
                }
                if (over) break;
                __threadfence_block();
                const int k = t.argq[j];
                const int v = t.rp[k];
                const uint32_t Eh = t.E[(size_t)t.rp[k - 1] * LT + gl];
                const bool light = (t.cstart[v + 1] - t.cstart[v]) > 1;
                if (light) build_G<LT>(c, t, w, v, gl, gmask);
                path_node<LT>(c, t, w, v, Eh, true, light, gl, gbase, gmask, nH, nV, opp, false, hmat(v));
            }
        }
    }
    __syncthreads();
    TMARK(3);
    // ---------------- backtrack: top-down path walks (S5)
    // The backtrack step of a node is a fixed map from its parent's span to its own span
    // (lt = smallest l of the span minimising E_v(l), R11; ls = recE_v(lt); span = recB_v(ls)).
    // All threads tabulate that map per node (spans as triangular codes, one byte per parent
    // span) into the dead leg-cost tables; a path walk is then one shared-memory byte load per
    // node, and the segment records are derived in the parallel output pass below.
    if constexpr (LT * (LT + 1) / 2 <= 8 * LT) {
        constexpr int NSP = LT * (LT + 1) / 2;
        constexpr int MSB = (NSP + 3) & ~3;   // map bytes per node (legH + legV give 8 LT per node)
        uint8_t* smap = reinterpret_cast<uint8_t*>(t.legH);
        auto code = [](int sp) -> int {        // (lo << 4 | hi) -> triangular code
            const int lo = sp >> 4, hi = sp & 15;
            return max(0, min(lo * (2 * LT - lo + 1) / 2 + (hi - lo), NSP - 1));
        };
        for (int v = 1 + tid; v < m; v += T) {
            uint32_t ev[LT], cs[LT];
#pragma unroll
            for (int l = 0; l < LT; l++) {
                ev[l] = t.E[(size_t)v * LT + l];
                cs[l] = (uint32_t)code(t.recB[(size_t)v * LT + t.recE[(size_t)v * LT + l]]);
            }
            uint32_t* out = reinterpret_cast<uint32_t*>(smap + (size_t)v * MSB);
            uint32_t word = 0;
            int idx = 0;
#pragma unroll
            for (int lo = 0; lo < LT; lo++) {
                uint32_t be = ev[lo], cc = cs[lo];
#pragma unroll
                for (int hi = lo; hi < LT; hi++) {
                    if (hi > lo && ev[hi] < be) { be = ev[hi]; cc = cs[hi]; }
                    word |= cc << (8 * (idx & 3));
                    if ((idx & 3) == 3) { out[idx >> 2] = word; word = 0; }
                    idx++;
                }
            }
            if (idx & 3) out[idx >> 2] = word;
        }
        if (tid == 0) t.span[0] = (uint8_t)code(t.span[0]);
        __syncthreads();
        // one lane per path; warps take paths by ticket, shallowest top first, so every
        // awaited path top's parent is held by a running warp (no deadlock)
        for (;;) {
            int p = 0;
            if (lane == 0) p = atomicAdd(&s_ticket2, 1);
            p = __shfl_sync(0xffffffffu, p, 0);
            if (p >= npaths) break;
            if (lane != 0) continue;
            const int tp = t.pq[npaths - 1 - p];
            int v, sp;
            if (tp == 0) { v = t.hv[0]; sp = t.span[0]; }
            else {
                const int u0 = t.par[tp];
                while (ld_flag(&t.sready[u0]) == 0) __nanosleep(32);
                __threadfence_block();
                v = tp;
                sp = t.span[u0];
            }
            while (v != 0xFFFF) {
                sp = smap[(size_t)v * MSB + sp];
                t.span[v] = (uint8_t)sp;
                if (t.cstart[v + 1] - t.cstart[v] > 1) {   // light children wait for this span
                    __threadfence_block();
                    *(volatile uint8_t*)&t.sready[v] = 1;
                }
                v = t.hv[v];
            }
        }
        __syncthreads();
        TMARK(4);
        TMARK(5);
        // segment records from the parent's span, outputs, and S6 for the whole net in one pass
        for (int i = 1 + tid; i < m; i += T) {
            const int u = t.par[i];
            const int cp = t.span[u];
            int lo = 0;
#pragma unroll
            for (int l = 1; l < LT; l++) lo += cp >= l * (2 * LT - l + 1) / 2 ? 1 : 0;
            const int hi = lo + cp - lo * (2 * LT - lo + 1) / 2;
            uint32_t be = 0xFFFFFFFFu;
            int lt = lo;
#pragma unroll
            for (int l = 0; l < LT; l++) {
                const uint32_t e = t.E[(size_t)i * LT + l];
                if (l >= lo && l <= hi && e < be) { be = e; lt = l; }   // smallest l attaining the min (R11)
            }
            const int ls = t.recE[(size_t)i * LT + lt];
            const bool straight = (t.x[i] == t.x[u]) || (t.y[i] == t.y[u]);
            const uint32_t s = seg_bend(h->dir[ls], h->dir[lt], straight) | ((uint32_t)ls << 8) | ((uint32_t)lt << 16) |
                               ((uint32_t)straight << 24);
            if (o.rec_seg) o.rec_seg[o.rec_off[o.list_base + idx] + i] = s;
            else o.seg[a0 + i] = s;
            if (commit) commit_edge(g, h, t.x[i], t.y[i], t.x[u], t.y[u], s, hyb_z(hy, a0 + i, s, LT));
        }
    } else {
        // ---------------- backtrack: top-down path walks (S5), one lane per path
        // A walk is a scalar chain (span of u -> lt -> ls -> span of v), so lane 0 of a warp
        // walks a path with the parent's span in a register (no shuffles, no per-node warp
        // synchronisation); a path whose top hangs off another path waits for that node's span
        // (sready).  Warps take paths by ticket, shallowest top first, so every awaited path is
        // already held by a running warp (no deadlock).
        for (;;) {
            int p = 0;
            if (lane == 0) p = atomicAdd(&s_ticket2, 1);
            p = __shfl_sync(0xffffffffu, p, 0);
            if (p >= npaths) break;
            if (lane != 0) continue;
            const int tp = t.pq[npaths - 1 - p];
            int v, sp;
            if (tp == 0) { v = t.hv[0]; sp = t.span[0]; }
            else {
                const int u0 = t.par[tp];
                while (ld_flag(&t.sready[u0]) == 0) __nanosleep(32);
                __threadfence_block();
                v = tp;
                sp = t.span[u0];
            }
            while (v != 0xFFFF) {
                const int u = t.par[v];
                const int lo = sp >> 4, hi = sp & 15;
                uint32_t ev[LT];
#pragma unroll
                for (int l = 0; l < LT; l++) ev[l] = t.E[(size_t)v * LT + l];
                uint32_t be = 0xFFFFFFFFu;
                int lt = lo;
#pragma unroll
                for (int l = 0; l < LT; l++)
                    if (l >= lo && l <= hi && ev[l] < be) { be = ev[l]; lt = l; }   // smallest l attaining the min (R11)
                const int ls = t.recE[(size_t)v * LT + lt];
                sp = t.recB[(size_t)v * LT + ls];
                t.span[v] = (uint8_t)sp;
                const bool straight = (t.x[v] == t.x[u]) || (t.y[v] == t.y[u]);
                const uint32_t bend = seg_bend(h->dir[ls], h->dir[lt], straight);
                t.legH[(size_t)v * 2 * nH] = bend | ((uint32_t)ls << 8) | ((uint32_t)lt << 16) | ((uint32_t)straight << 24);
                if (t.cstart[v + 1] - t.cstart[v] > 1) {   // light children wait for this span
                    __threadfence_block();
                    *(volatile uint8_t*)&t.sready[v] = 1;
                }
                v = t.hv[v];
            }
        }
        __syncthreads();
        TMARK(4);
        TMARK(5);
        // outputs and S6 for the whole net in one pass (the atomics' latencies overlap across threads)
        for (int i = 1 + tid; i < m; i += T) {
            const uint32_t s = t.legH[(size_t)i * 2 * nH];
            if (o.rec_seg) o.rec_seg[o.rec_off[o.list_base + idx] + i] = s;
            else o.seg[a0 + i] = s;
            if (commit) {
                const int u = t.par[i];
                commit_edge(g, h, t.x[i], t.y[i], t.x[u], t.y[u], s, hyb_z(hy, a0 + i, s, LT));
            }
        }
    }
#ifdef FGR_TIMING
    __syncthreads();
    TMARK(6);
    if (tid == 0 && m > 600)
        printf("TIMING m=%d maxd=%d paths=%d prologue=%lld gather=%lld dp=%lld backtrack=%lld commit=%lld\n", m, K - 1,
               npaths, tm[1] - tm[0], tm[2] - tm[1], tm[3] - tm[2], tm[4] - tm[3], tm[6] - tm[5]);
#endif
    if (tid == 0) {
        const uint32_t total = (uint32_t)(s_root >> 8);
        if (o.rec_seg) { o.rec_seg[o.rec_off[o.list_base + idx]] = 0xFFFFFFFFu; o.rec_cost[o.list_base + idx] = total; }
        else { o.seg[a0] = 0xFFFFFFFFu; o.cost[net] = total; }
    }
}

// One CTA per large net: the demand-independent tree analysis, written to global memory once per stage.
// Only the analysis arrays live in shared memory (~38 B/node, not the DP tables), and 256
// threads at <= 64 registers, so several nets share an SM.
constexpr int kPrepThreads = 256;

__host__ __device__ inline size_t prep_bytes(int m) {
    return 2 * a16((size_t)(m + 1) * 4) + 11 * a16((size_t)m * 2) + 2 * a16((size_t)(m + 1) * 2) + 4 * a16((size_t)m);
}

__device__ inline Tabs carve_prep(unsigned char* p, int m) {
    Tabs t;
    t.E = nullptr; t.aux = nullptr; t.recE = nullptr; t.recB = nullptr; t.span = nullptr; t.rp = nullptr; t.argq = nullptr;
    auto u16 = [&](size_t n) { uint16_t* q = (uint16_t*)p; p += a16(n * 2); return q; };
    t.legH = (uint32_t*)p; p += a16((size_t)(m + 1) * 4);   // child counts (scratch)
    t.legV = (uint32_t*)p; p += a16((size_t)(m + 1) * 4);   // level counts (scratch)
    t.x = (int16_t*)u16(m); t.y = (int16_t*)u16(m); t.par = (int16_t*)u16(m); t.depth = u16(m);
    t.anc = u16(m); t.hv = u16(m); t.top = u16(m); t.bot = u16(m); t.pq = u16(m); t.rpos = u16(m); t.clist = u16(m);
    t.cstart = u16(m + 1); t.lvstart = u16(m + 1);
    t.done = p; p += a16((size_t)m);
    t.sready = p; p += a16((size_t)m);
    t.plo = (int8_t*)p; p += a16((size_t)m);
    t.phi = (int8_t*)p;
    return t;
}

template <int LT>
__global__ void __launch_bounds__(kPrepThreads, 4) k_large_prep(GridView g, NetsView nv, const int32_t* __restrict__ list,
                                                                 uint16_t* cs, uint16_t* cl, uint16_t* hv, uint16_t* bot,
                                                                 uint16_t* pq, uint16_t* rpos, int32_t* npaths) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ int s_maxd, s_npaths, s_deep;
    if (threadIdx.x == 0) { s_maxd = 0; s_npaths = 0; }
    const int warp = threadIdx.x >> 5, lane = lane_id(), tid = threadIdx.x, T = blockDim.x;
    const int net = list[blockIdx.x];
    const int a0 = nv.off[net];
    const int m = nv.off[net + 1] - a0;
    const Tabs t = carve_prep(smem, m);
    large_prologue(t, nv, a0, m, tid, T, warp, lane, &s_maxd, &s_npaths, &s_deep);
    __syncthreads();
    for (int i = tid; i < m; i += T) {
        cs[a0 + i] = t.cstart[i]; cl[a0 + i] = t.clist[i]; hv[a0 + i] = t.hv[i];
        bot[a0 + i] = t.bot[i]; pq[a0 + i] = t.pq[i]; rpos[a0 + i] = t.rpos[i];
    }
    if (tid == 0) npaths[net] = s_npaths;
}

// ------------------------------------------------------------- thread kernel (2-node nets)
// Half of all nets have one tree edge.  One thread routes one such net with the
// whole DP in registers: leaf B(ls) and the root minimum in the closed form of
// G for K = V (no light children), the edge step of Eqs. (1),(3),(5)-(7) over
// both bends, the R11 tie-breaks, the backtrack and the commit.
constexpr int kTwoThreads = 128;

// leg costs for one leg into a transposed per-thread scratch column (stride kTwoThreads)
__device__ __forceinline__ void leg_cost_col(const DirView& d, int line, int a, int b, uint32_t* col) {
    const size_t pa = ((size_t)line * d.len + a) * d.W, pb = ((size_t)line * d.len + b) * d.W;
    const size_t sa = ((size_t)line * d.nseg + (a >> FGR_SEG_SHIFT)) * d.W;
    const size_t sb = ((size_t)line * d.nseg + (b >> FGR_SEG_SHIFT)) * d.W;
    const int nq = d.W >> 2;
#pragma unroll
    for (int q = 0; q < 4; q++) {
        if (q < nq) {
            const uint4 Pa = __ldg(reinterpret_cast<const uint4*>(d.P + pa) + q);
            const uint4 Pb = __ldg(reinterpret_cast<const uint4*>(d.P + pb) + q);
            uint4 Sa = make_uint4(0, 0, 0, 0), Sb = Sa;
            if (sa != sb) {   // inside one segment the bases cancel
                Sa = __ldg(reinterpret_cast<const uint4*>(d.SB + sa) + q);
                Sb = __ldg(reinterpret_cast<const uint4*>(d.SB + sb) + q);
            }
            col[(4 * q + 0) * kTwoThreads] = (Sb.x + Pb.x) - (Sa.x + Pa.x);
            col[(4 * q + 1) * kTwoThreads] = (Sb.y + Pb.y) - (Sa.y + Pa.y);
            col[(4 * q + 2) * kTwoThreads] = (Sb.z + Pb.z) - (Sa.z + Pa.z);
            col[(4 * q + 3) * kTwoThreads] = (Sb.w + Pb.w) - (Sa.w + Pa.w);
        }
    }
}

template <int LT>
__global__ void __launch_bounds__(kTwoThreads) k_dp_two(GridView g, NetsView nv, const int32_t* __restrict__ list,
                                                        int count, Out o, int commit, HybView hy) {
    __shared__ Hdr hs;
    __shared__ uint32_t legs[4 * 16 * kTwoThreads];   // [leg][slot][thread]
    init_hdr(&hs, g);
    __syncthreads();
    const int tid = threadIdx.x;
    const int idx = blockIdx.x * kTwoThreads + tid;
    if (idx >= count) return;
    uint32_t vp[LT], zl[LT], sl[LT];
    uint32_t hmask = 0;
#pragma unroll
    for (int l = 0; l < LT; l++) {
        vp[l] = hs.viapre[l]; zl[l] = hs.zlo[l]; sl[l] = hs.slot[l];
        hmask |= (hs.dir[l] == 0 ? 1u : 0u) << l;
    }
    const int net = list[idx];
    const int a0 = nv.off[net];
    if (nv.off[net + 1] - a0 < 2) {   // trivial net: no edge, cost 0
        if (o.rec_seg) { o.rec_seg[o.rec_off[o.list_base + idx]] = 0xFFFFFFFFu; o.rec_cost[o.list_base + idx] = 0; }
        else { o.seg[a0] = 0xFFFFFFFFu; o.cost[net] = 0; }
        return;
    }
    const int x0 = nv.x[a0], y0 = nv.y[a0], x1 = nv.x[a0 + 1], y1 = nv.y[a0 + 1];
    const int hslot = hy.net ? hy.net[net] : -1;   // a 2-node net's first slot is its only edge
    const int plo0 = nv.plo[a0], phi0 = nv.phi[a0], plo1 = nv.plo[a0 + 1], phi1 = nv.phi[a0 + 1];
    const bool sh = (y0 == y1), sv = (x0 == x1), straight = sh || sv;
    uint32_t* col = legs + tid;
    // legs: 0 = H row y1, 1 = H row y0, 2 = V col x1, 3 = V col x0   (x1..x0 / y1..y0)
    const int xa = min(x0, x1), xb = max(x0, x1), ya = min(y0, y1), yb = max(y0, y1);
    if (!sv) leg_cost_col(g.h, y1, xa, xb, col + 0 * 16 * kTwoThreads);
    if (!straight) leg_cost_col(g.h, y0, xa, xb, col + 1 * 16 * kTwoThreads);
    if (!sh) leg_cost_col(g.v, x1, ya, yb, col + 2 * 16 * kTwoThreads);
    if (!straight) leg_cost_col(g.v, x0, ya, yb, col + 3 * 16 * kTwoThreads);
    uint32_t c1[LT], c2[LT];   // leg 1 on layer l (from the leaf), leg 2 on layer l (into the root)
#pragma unroll
    for (int l = 0; l < LT; l++) {
        const bool hl = (hmask >> l) & 1u;
        c1[l] = col[((hl ? 0 : 2) * 16 + sl[l]) * kTwoThreads];
        c2[l] = straight ? 0u : col[((hl ? 1 : 3) * 16 + sl[l]) * kTwoThreads];
    }
    // leaf: B(ls) = G(a, b), a = min(ls, pin_lo), b = max(ls, pin_hi), closed form (K = V)
    uint32_t vplo = 0, vphi = 0, zplo = 0;
#pragma unroll
    for (int l = 0; l < LT; l++) {
        vplo = (l == plo1) ? vp[l] : vplo;
        vphi = (l == phi1) ? vp[l] : vphi;
        zplo = (l == plo1) ? zl[l] : zplo;
    }
    uint32_t Bv[LT];
    uint8_t recB[LT];
#pragma unroll
    for (int ls = 0; ls < LT; ls++) {
        uint32_t va, vb, za, bb;
        if (plo1 >= 0) {
            va = ls <= plo1 ? vp[ls] : vplo;
            za = ls <= plo1 ? zl[ls] : zplo;
            vb = ls >= phi1 ? vp[ls] : vphi;
            bb = ls >= phi1 ? (uint32_t)ls : (uint32_t)phi1;
        } else {
            va = vb = vp[ls]; za = zl[ls]; bb = ls;
        }
        Bv[ls] = vb - va;
        recB[ls] = (uint8_t)((za << 4) | bb);
    }
    // edge: E(lt), recE(lt)
    uint32_t E[LT];
    uint8_t recE[LT];
    const int de = sh ? 0 : 1;
#pragma unroll
    for (int lt = 0; lt < LT; lt++) {
        const bool hlt = (hmask >> lt) & 1u;
        uint32_t best = FGR_INF;
        int bls = lt;
        if (hslot >= 0) {   // hybrid edge: min-plus with the precomputed transfer matrix
            const uint32_t* hm = hy.M + ((size_t)hslot * LT + lt) * LT;
#pragma unroll
            for (int ls = 0; ls < LT; ls++) {
                const uint32_t cst = sat_add(Bv[ls], hm[ls]);
                if (cst < best) { best = cst; bls = ls; }
            }
        } else if (straight) {
            if ((hlt ? 0 : 1) == de) best = sat_add(Bv[lt], c1[lt]);
        } else {
#pragma unroll
            for (int ls = 0; ls < LT; ls++) {
                const bool hls = (hmask >> ls) & 1u;
                if (hls != hlt) {
                    const uint32_t via = vp[ls] > vp[lt] ? vp[ls] - vp[lt] : vp[lt] - vp[ls];
                    const uint32_t cst = sat_add(sat_add(sat_add(Bv[ls], c1[ls]), via), c2[lt]);
                    if (cst < best) { best = cst; bls = ls; }
                }
            }
        }
        E[lt] = best;
        recE[lt] = (uint8_t)bls;
    }
    // root, generalised Eq. (4): min over l of E(l) + G(hull({l} + pins))
    uint32_t vrlo = 0, vrhi = 0, zrlo = 0;
#pragma unroll
    for (int l = 0; l < LT; l++) {
        vrlo = (l == plo0) ? vp[l] : vrlo;
        vrhi = (l == phi0) ? vp[l] : vrhi;
        zrlo = (l == plo0) ? zl[l] : zrlo;
    }
    unsigned long long kk[LT];
#pragma unroll
    for (int l = 0; l < LT; l++) {
        uint32_t va, vb, za, bb;
        if (plo0 >= 0) {
            va = l <= plo0 ? vp[l] : vrlo;
            za = l <= plo0 ? zl[l] : zrlo;
            vb = l >= phi0 ? vp[l] : vrhi;
            bb = l >= phi0 ? (uint32_t)l : (uint32_t)phi0;
        } else {
            va = vb = vp[l]; za = zl[l]; bb = l;
        }
        kk[l] = ((unsigned long long)sat_add(E[l], vb - va) << 8) | (za << 4) | bb;
    }
    const unsigned long long rk = tree_min<LT>(kk);
    // backtrack: lt = smallest layer in the root span minimising E (R11)
    const int lo = (int)((rk >> 4) & 15), hi = (int)(rk & 15);
    uint32_t be = FGR_INF + 1u;
    int lt = lo, ls = lo;
#pragma unroll
    for (int l = 0; l < LT; l++)
        if (l >= lo && l <= hi && E[l] < be) { be = E[l]; lt = l; ls = recE[l]; }
    (void)recB;
    const uint32_t bend = seg_bend(((hmask >> ls) & 1u) ? 0 : 1, ((hmask >> lt) & 1u) ? 0 : 1, straight);
    const uint32_t sg = bend | ((uint32_t)ls << 8) | ((uint32_t)lt << 16) | ((uint32_t)(straight ? 1 : 0) << 24);
    if (o.rec_seg) {
        uint32_t* rs = o.rec_seg + o.rec_off[o.list_base + idx];
        rs[0] = 0xFFFFFFFFu; rs[1] = sg;
        o.rec_cost[o.list_base + idx] = (uint32_t)(rk >> 8);
    } else {
        o.seg[a0] = 0xFFFFFFFFu; o.seg[a0 + 1] = sg;
        o.cost[net] = (uint32_t)(rk >> 8);
    }
    if (commit) commit_edge(g, &hs, x1, y1, x0, y0, sg, hyb_z(hy, a0 + 1, sg, LT));
}

// Commit from route records (multi-GPU: after the exchange every rank commits every net).
__global__ void __launch_bounds__(256) k_commit_records(GridView g, NetsView nv, const int32_t* __restrict__ list, int count,
                                                        const uint32_t* __restrict__ rec_seg,
                                                        const int32_t* __restrict__ rec_off, int list_base, HybView hy) {
    __shared__ Hdr hs;
    init_hdr(&hs, g);
    __syncthreads();
    const int warp = (int)((blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5);
    const int nwarps = (int)((gridDim.x * (size_t)blockDim.x) >> 5);
    for (int idx = warp; idx < count; idx += nwarps) {
        const int net = list[idx];
        const int a0 = nv.off[net], m = nv.off[net + 1] - a0;
        const uint32_t* rs = rec_seg + rec_off[list_base + idx];
        for (int i = 1 + lane_id(); i < m; i += 32) {
            const int u = nv.par[a0 + i];
            commit_edge(g, &hs, nv.x[a0 + i], nv.y[a0 + i], nv.x[a0 + u], nv.y[a0 + u], rs[i], hyb_z(hy, a0 + i, rs[i], g.L));
        }
    }
}

// ------------------------------------------------------------- host side
size_t smem_large(int L, int nH, int nV, int m) {
    return a16(sizeof(Hdr)) + (size_t)kLargeWarps * wscr_bytes(L) + tabs_bytes(m, L, nH, nV, true) +
           (size_t)kMR * L * ((L + 3) & ~3) * 4;
}

}  // namespace

// Largest net the shared-memory heavy-path kernel (k_dp_large) holds; bigger nets take k_dp_hld.
int fgr_large_limit(const fgr_grid* g) {
    int m = 2048;
    while (m > FGR_SMALL_NET && smem_large(g->L, g->nH, g->nV, m) + 64 > (size_t)g->max_smem) m -= 16;
    return m;
}

// Largest net routed by a shared-memory kernel under the grid's DP policy (k_dp_tree for
// FGR_DP_AUTO, k_dp_large for FGR_DP_HEAVY); bigger nets take k_dp_hld.
int fgr_top_limit(const fgr_grid* g) {
    return g->dp_policy == FGR_DP_AUTO ? fgr_tree_cap(g) : fgr_large_limit(g);
}

namespace {

template <int LT>
cudaError_t launch_lt(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int nlarge, int nmidL,
                      int nmidS, int ntwo, int maxm_large, const Out& o, bool commit, const Prep& prep,
                      const int* lsplit) {
    static bool configured = false;   // one device per process is the supported configuration
    if (!configured) {
        cudaFuncAttributes fa;
        cudaError_t e = cudaFuncGetAttributes(&fa, k_dp_large<LT>);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(k_dp_large<LT>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     g->max_smem - (int)fa.sharedSizeBytes);
        if (e == cudaSuccess) e = cudaFuncGetAttributes(&fa, k_large_prep<LT>);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(k_large_prep<LT>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     g->max_smem - (int)fa.sharedSizeBytes);
        if (e != cudaSuccess) return e;
        configured = true;
    }
    const GridView& v = g->view;
    const HybView hyv = g->hy.view();
    // Launch units: large-net size buckets (the list is in descending size): above the heavy-path
    // kernel's shared-memory limit, then > 512, 257..512, 129..256, 65..128, 33..64 nodes (one bucket
    // unless lsplit is given), then the classes 9..32, 3..8 and 2 nodes.  Units are independent nets:
    // each non-empty unit gets its own stream (forked from and joined back into the caller's stream).
    const int lim = fgr_top_limit(g);
    const bool tree = g->dp_policy == FGR_DP_AUTO;
    struct Unit { int kind, off, n, cap; };   // kind: 0 large, 1 midL, 2 midS, 3 two
    Unit units[10];
    int nu = 0;
    {
        // thresholds (descending) with the number of large nets above each; the tree kernel
        // (FGR_DP_AUTO) takes three buckets: (512, lim], (128, 512], (32, 128]
        int thr[5] = {lim, 512, 256, 128, 64}, above[5] = {0, 0, 0, 0, 0};
        bool use[5] = {true, true, !tree, true, !tree};
        if (lsplit) for (int k = 0; k < 5; k++) above[k] = min(lsplit[k], nlarge);
        for (int i = 0; i < 5; i++)
            for (int j = i + 1; j < 5; j++)
                if (thr[j] > thr[i]) {
                    int x = thr[i]; thr[i] = thr[j]; thr[j] = x; x = above[i]; above[i] = above[j]; above[j] = x;
                    bool y = use[i]; use[i] = use[j]; use[j] = y;
                }
        int prev = 0, cap = maxm_large;
        for (int k = 0; k <= 5 && prev < nlarge; k++) {
            if (k < 5 && !use[k]) continue;
            const int end = (k < 5 && lsplit) ? max(prev, above[k]) : nlarge;
            if (end > prev) units[nu++] = Unit{0, prev, end - prev, min(cap, maxm_large)};
            prev = end;
            if (k < 5) cap = thr[k];
        }
    }
    if (nmidL > 0) units[nu++] = Unit{1, nlarge, nmidL, 0};
    if (nmidS > 0) units[nu++] = Unit{2, nlarge + nmidL, nmidS, 0};
    if (ntwo > 0) units[nu++] = Unit{3, nlarge + nmidL + nmidS, ntwo, 0};
    // kernel of a large-net unit (fgr_set_dp_policy): the contraction kernel above lim or under
    // FGR_DP_HLD; FGR_DP_AUTO: the tree kernel; FGR_DP_HEAVY: the dataflow kernel up to flow_max
    // nodes, then the heavy-path kernel
    auto large_kind = [&](int cap) {   // 0 hld, 1 flow, 2 heavy-path, 3 tree
        if (cap > lim || g->dp_policy == FGR_DP_HLD) return 0;
        if (tree) return 3;
        if (cap <= g->flow_max && cap <= fgr_flow_max_nodes(g)) return 1;
        return 2;
    };
    const bool fork = nu > 1;
    cudaError_t e;
    int tree_off = 0, tree_n = 0, tree_cap = 0;   // the tree-kernel units (contiguous in the list) share one commit
    // global workspaces of the large-net units (one region each: the units run concurrently)
    size_t wsoff[10] = {0}, wstot = 0;
    unsigned char* wsb = nullptr;
    {
        for (int ui = 0; ui < nu; ui++) {
            if (units[ui].kind != 0) continue;
            const int lk = large_kind(units[ui].cap);
            // k_dp_hld: per-CTA workspaces; tree units above 128 nodes: their nets' leg rows (k_tree_legs)
            const size_t b = lk == 0 ? fgr_hld_ws_bytes(g, units[ui].n, units[ui].cap)
                             : (lk == 3 && units[ui].cap > 128) ? (size_t)units[ui].n * 2 * units[ui].cap * LT * 4 : 0;
            wsoff[ui] = wstot;
            wstot += (b + 255) & ~(size_t)255;
        }
        if (wstot > 0) {
            wsb = (unsigned char*)fgr_scratch(g->s_hldw, wstot, &e);
            if (e != cudaSuccess) return e;
        }
    }
    if (fork) {
        // recorded before any launch: the side streams wait for the refresh, not for each other
        if ((e = cudaEventRecord(g->ev_fork, st)) != cudaSuccess) return e;
        for (int i = 0; i + 1 < nu; i++)
            if ((e = cudaStreamWaitEvent(g->side[i], g->ev_fork, 0)) != cudaSuccess) return e;
    }
    for (int ui = 0; ui < nu; ui++) {
        const Unit& un = units[ui];
        cudaStream_t su = ui == 0 ? st : g->side[ui - 1];
        Out os = o;
        os.list_base = o.list_base + un.off;
        const int32_t* l = list + un.off;
        const int n = un.n;
        const int ps = fgr_prof_begin(g, un.kind == 0 ? PROF_DP_LARGE : PROF_DP_SMALL, su);
        const int lk = un.kind == 0 ? large_kind(un.cap) : -1;
        if (lk == 0) {
            e = fgr_launch_hld(g, su, nv, l, n, un.cap, os, commit, prep.hld, wsb ? wsb + wsoff[ui] : nullptr);
            if (e != cudaSuccess) return e;
        } else if (lk == 3) {
            uint32_t* legs = nullptr;   // nets above 128 nodes: leg costs gathered by many SMs first
            if (un.cap > 128) {
                legs = reinterpret_cast<uint32_t*>(wsb + wsoff[ui]);   // this unit's own region (units run concurrently)
                if ((e = fgr_launch_tree_legs(g, su, nv, l, n, un.cap, legs)) != cudaSuccess) return e;
            }
            e = fgr_launch_tree(g, su, nv, l, n, un.cap, os, false, prep.hld, legs, un.cap);   // committed after the join
            if (tree_n == 0) { tree_off = un.off; tree_cap = un.cap; }
            tree_n += n;
            if (e != cudaSuccess) return e;
        } else if (lk == 1) {
            e = fgr_launch_flow(g, su, nv, l, n, un.cap, os, commit, prep);
            if (e != cudaSuccess) return e;
        } else if (un.kind == 0) {
            // programmatic dependent launch: the prologue overlaps the refresh that precedes it
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(n);
            cfg.blockDim = dim3(32 * kLargeWarps);
            cfg.dynamicSmemBytes = smem_large(LT, g->nH, g->nV, un.cap);
            cfg.stream = su;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
            at[0].val.programmaticStreamSerializationAllowed = 1;
            cfg.attrs = at;
            cfg.numAttrs = 1;
            e = cudaLaunchKernelEx(&cfg, k_dp_large<LT>, v, nv, l, n, os, commit ? 1 : 0, prep, hyv);
            if (e != cudaSuccess) return e;
        } else if (un.kind <= 2) {
            e = fgr_launch_walk(g, su, nv, l, n, un.kind == 1 ? FGR_SMALL_NET : FGR_MID_NET, os, commit);
            if (e != cudaSuccess) return e;
        } else {
            k_dp_two<LT><<<(n + kTwoThreads - 1) / kTwoThreads, kTwoThreads, 0, su>>>(v, nv, l, n, os, commit ? 1 : 0,
                                                                                      hyv);
        }
        fgr_prof_end(g, ps, su);
        g->stats.kernel_launches++;
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
    }
    if (fork) {
        for (int i = 0; i + 1 < nu; i++) {
            if ((e = cudaEventRecord(g->ev_join[i], g->side[i])) != cudaSuccess) return e;
            if ((e = cudaStreamWaitEvent(st, g->ev_join[i], 0)) != cudaSuccess) return e;
        }
    }
    if (commit && tree_n > 0) {
        Out os = o;
        os.list_base = o.list_base + tree_off;
        const int ps = fgr_prof_begin(g, PROF_COMMIT, st);
        e = fgr_launch_commit_nets(g, st, nv, list + tree_off, tree_n, tree_cap, os);
        fgr_prof_end(g, ps, st);
        if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
}

}  // namespace


size_t fgr_dp_smem_large(const fgr_grid* g, int m) { return smem_large(g->L, g->nH, g->nV, m); }

cudaError_t fgr_launch_dp(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int nlarge, int nmidL,
                          int nmidS, int ntwo, int maxm_large, uint32_t* seg_out, uint32_t* cost_out, uint32_t* rec_seg,
                          const int32_t* rec_off, uint32_t* rec_cost, int list_base, bool commit, const Prep* prep,
                          const int* lsplit) {
    const Prep pz = {};
    const Prep& pp = prep ? *prep : pz;
    Out o;
    o.seg = seg_out; o.cost = cost_out; o.rec_seg = rec_seg; o.rec_off = rec_off; o.rec_cost = rec_cost;
    o.list_base = list_base;
    switch (g->L) {
#define FGR_LT(n) case n: return launch_lt<n>(g, st, nv, list, nlarge, nmidL, nmidS, ntwo, maxm_large, o, commit, pp, lsplit);
        FGR_LT(2) FGR_LT(3) FGR_LT(4) FGR_LT(5) FGR_LT(6) FGR_LT(7) FGR_LT(8) FGR_LT(9) FGR_LT(10) FGR_LT(11)
        FGR_LT(12) FGR_LT(13) FGR_LT(14) FGR_LT(15) FGR_LT(16)
#undef FGR_LT
        default: return cudaErrorInvalidValue;
    }
}

namespace {
template <int LT>
cudaError_t launch_prep_lt(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int count, int maxm,
                           uint16_t* cs, uint16_t* cl, uint16_t* hv, uint16_t* bot, uint16_t* pq, uint16_t* rpos,
                           int32_t* np) {
    cudaFuncAttributes fa;
    cudaError_t e = cudaFuncGetAttributes(&fa, k_large_prep<LT>);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_large_prep<LT>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 g->max_smem - (int)fa.sharedSizeBytes);
    if (e != cudaSuccess) return e;
    k_large_prep<LT><<<count, kPrepThreads, prep_bytes(maxm), st>>>(g->view, nv, list, cs, cl, hv, bot, pq, rpos, np);
    g->stats.kernel_launches++;
    return cudaGetLastError();
}
}  // namespace

cudaError_t fgr_launch_large_prep(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int count,
                                  int maxm, uint16_t* cs, uint16_t* cl, uint16_t* hv, uint16_t* bot, uint16_t* pq,
                                  uint16_t* rpos, int32_t* np) {
    if (count <= 0) return cudaSuccess;
    switch (g->L) {
#define FGR_LT(n) case n: return launch_prep_lt<n>(g, st, nv, list, count, maxm, cs, cl, hv, bot, pq, rpos, np);
        FGR_LT(2) FGR_LT(3) FGR_LT(4) FGR_LT(5) FGR_LT(6) FGR_LT(7) FGR_LT(8) FGR_LT(9) FGR_LT(10) FGR_LT(11)
        FGR_LT(12) FGR_LT(13) FGR_LT(14) FGR_LT(15) FGR_LT(16)
#undef FGR_LT
        default: return cudaErrorInvalidValue;
    }
}

cudaError_t fgr_launch_commit(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int count,
                              const uint32_t* rec_seg, const int32_t* rec_off, int list_base) {
    const GridView& v = g->view;
    int blocks = (count + 7) / 8;
    if (blocks > g->num_sms * 8) blocks = g->num_sms * 8;
    if (blocks < 1) blocks = 1;
    const int ps = fgr_prof_begin(g, PROF_COMMIT, st);
    k_commit_records<<<blocks, 256, 0, st>>>(v, nv, list, count, rec_seg, rec_off, list_base, g->hy.view());
    fgr_prof_end(g, ps, st);
    g->stats.kernel_launches++;
    return cudaGetLastError();
}
