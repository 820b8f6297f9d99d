// dp_walk.cu — the tree DP (S4), backtrack (S5) and commit (S6) for nets with 3..32
// nodes: one lane group per net, LT lanes per group (lane = layer), G groups per warp
// walking their nets' nodes children-first in lockstep.
//
// Same recurrences as dp.cu (§III-D; readings R3, R5-R11), written
// for a short instruction path per node:
//   * node step, Eq. (2) by span enumeration (R3): lane lo builds the row
//       K(lo, hi) = V(lo, hi) + sum_c min_{l in [lo, hi]} E_c(l)      (hi >= lo)
//     and its suffix minima S(lo, b) = min_{hi >= b} K(lo, hi) with the smallest
//     attaining hi; lane ls then reads B_v(ls) = min_{lo <= a} S(lo, b) (a = min(ls,
//     pin_lo), b = max(ls, pin_hi)) taking the smallest attaining lo.  That is exactly
//     R11's (value, lo, hi) order on the spans, with 32-bit values and byte argmins.
//   * edge step, Eqs. (1), (3), (5)-(7) with both bends (R5): lane ls publishes
//     w1(ls) = B_v(ls) + leg1(ls); lane lt takes min_ls [w1(ls) + V(ls, lt)] over the
//     layers of the other direction (smallest ls on ties, R11) and adds its leg 2.
//     Leg costs are stored per lane column: LA = the leg on the child's line (row y_v
//     for an H lane, column x_v for a V lane), LB = the leg on the parent's line, so
//     bend 0 (ls in H) is leg1 = LA(ls), leg2 = LB(lt), and bend 1 is the same formula
//     with the directions swapped.
//   * root: generalised Eq. (4) (R9), the same lookup with a = pin_lo, b = pin_hi
//     (a = L-1, b = 0 for a Steiner root: any span).
//   * backtrack: one lane per net, ascending node index (parents first, R22).
#include "dp_common.cuh"

namespace {

template <int LT>
struct WK {
    static constexpr int ES = (LT + 3) & ~3;   // words per per-layer row (16-byte rows)
    static constexpr int G = groups_of(LT);
};

struct WHdr {
    Hdr h;
    uint8_t los[2][FGR_MAXL];   // layer of slot, per direction
};

struct WTabs {                  // one net's tables in shared memory
    uint32_t* E;    // [mc][ES]  E_v(lt)
    uint32_t* LA;   // [mc][ES]  leg on the child's line, per layer
    uint32_t* LB;   // [mc][ES]  leg on the parent's line, per layer
    uint32_t* S;    // [LT][ES]  scratch: suffix minima rows
    uint32_t* BW;   // [2][ES]   scratch: B_v, w1
    uint32_t* cm;   // [mc]      children bitmask
    uint32_t* seg;  // [mc]      chosen route (backtrack)
    uint8_t* recE;  // [mc][ES]  argmin ls of E_v(lt)
    uint8_t* recB;  // [mc][ES]  argmin span (lo << 4 | hi) of B_v(ls)
    uint8_t* HA;    // [LT][ES]  scratch: argmin hi of the suffix minima
    int16_t* x;
    int16_t* y;
    uint16_t* par;
    int8_t* plo;
    int8_t* phi;
    uint8_t* span;
};

__host__ __device__ inline size_t wtabs_bytes(int mc, int L) {
    const size_t ES = (size_t)((L + 3) & ~3);
    return 3 * a16(mc * ES * 4) + a16(L * ES * 4) + a16(2 * ES * 4) + 2 * a16((size_t)mc * 4) + 2 * a16(mc * ES) +
           a16(L * ES) + 3 * a16((size_t)mc * 2) + 3 * a16((size_t)mc);
}

__device__ inline WTabs carve_w(unsigned char* p, int mc, int L) {
    const size_t ES = (size_t)((L + 3) & ~3);
    WTabs t;
    t.E = (uint32_t*)p; p += a16(mc * ES * 4);
    t.LA = (uint32_t*)p; p += a16(mc * ES * 4);
    t.LB = (uint32_t*)p; p += a16(mc * ES * 4);
    t.S = (uint32_t*)p; p += a16(L * ES * 4);
    t.BW = (uint32_t*)p; p += a16(2 * ES * 4);
    t.cm = (uint32_t*)p; p += a16((size_t)mc * 4);
    t.seg = (uint32_t*)p; p += a16((size_t)mc * 4);
    t.recE = p; p += a16(mc * ES);
    t.recB = p; p += a16(mc * ES);
    t.HA = p; p += a16(L * ES);
    t.x = (int16_t*)p; p += a16((size_t)mc * 2);
    t.y = (int16_t*)p; p += a16((size_t)mc * 2);
    t.par = (uint16_t*)p; p += a16((size_t)mc * 2);
    t.plo = (int8_t*)p; p += a16((size_t)mc);
    t.phi = (int8_t*)p; p += a16((size_t)mc);
    t.span = p;
    return t;
}

// Per-lane constants of the lane that owns layer gl.
template <int LT>
struct WLane {
    uint32_t vrow[LT];   // V(gl, hi) for hi >= gl, INF below: the K row of lo = gl before the children
    uint32_t vmeo[LT];   // V(ls, gl) for ls of the other direction, INF for ls of gl's direction
    int my_dir;
    __device__ __forceinline__ void load(const Hdr* h, int gl) {
        const int me = gl < LT ? gl : 0;
        const uint32_t vm = h->viapre[me];
        my_dir = h->dir[me];
#pragma unroll
        for (int i = 0; i < LT; i++) {
            const uint32_t vi = h->viapre[i];
            vrow[i] = i >= me ? vi - vm : FGR_INF;
            vmeo[i] = h->dir[i] != my_dir ? (vi >= vm ? vi - vm : vm - vi) : FGR_INF;
        }
    }
};

// One node of the walk for the lane group (all lanes of the warp call it: the syncs are
// full-warp).  Non-root: writes E_v / recE_v / recB_v.  Root: writes span[0], *rootcost.
template <int LT, bool CSR>
__device__ __forceinline__ void wstep(const WLane<LT>& c, const WTabs& t, int v, bool act, bool root, int gl,
                                      const uint32_t* hm, uint32_t* rootcost, const uint16_t* cs = nullptr,
                                      const uint16_t* cl = nullptr) {
    constexpr int ES = WK<LT>::ES;
    // K row of lo = gl (F_v restricted to spans starting at gl)
    uint32_t acc[LT];
#pragma unroll
    for (int hi = 0; hi < LT; hi++) acc[hi] = c.vrow[hi];
    uint32_t cmask = (!CSR && act) ? t.cm[v] : 0u;
    int ck = 0, ce = 0;
    if (CSR && act) { ck = cs[v]; ce = cs[v + 1]; }
    while (CSR ? ck < ce : cmask != 0u) {
        int ch;
        if (CSR) ch = cl[ck++];
        else { ch = __ffs(cmask) - 1; cmask &= cmask - 1; }
        const uint4* ep = reinterpret_cast<const uint4*>(t.E + ch * ES);
        uint32_t e[ES];
#pragma unroll
        for (int q = 0; q < ES / 4; q++) {
            const uint4 w = ep[q];
            e[4 * q] = w.x; e[4 * q + 1] = w.y; e[4 * q + 2] = w.z; e[4 * q + 3] = w.w;
        }
        uint32_t run = FGR_INF;
#pragma unroll
        for (int hi = 0; hi < LT; hi++) {
            run = min(run, hi >= gl ? e[hi] : FGR_INF);
            acc[hi] = sat_add(acc[hi], run);
        }
    }
    // suffix minima over hi, ties keep the smaller hi
    uint32_t srow[ES], hp[ES / 4];
#pragma unroll
    for (int q = 0; q < ES / 4; q++) hp[q] = 0;
#pragma unroll
    for (int hi = LT; hi < ES; hi++) srow[hi] = FGR_INF;
    {
        uint32_t s = FGR_INF, ah = LT - 1;
#pragma unroll
        for (int hi = LT - 1; hi >= 0; hi--) {
            if (acc[hi] <= s) { s = acc[hi]; ah = (uint32_t)hi; }
            srow[hi] = s;
            hp[hi >> 2] |= ah << (8 * (hi & 3));
        }
    }
    if (act) {
        uint4* sp = reinterpret_cast<uint4*>(t.S + gl * ES);
        uint32_t* hpp = reinterpret_cast<uint32_t*>(t.HA + gl * ES);
#pragma unroll
        for (int q = 0; q < ES / 4; q++) {
            sp[q] = make_uint4(srow[4 * q], srow[4 * q + 1], srow[4 * q + 2], srow[4 * q + 3]);
            hpp[q] = hp[q];
        }
    }
    __syncwarp();
    // B_v(ls) for ls = gl (or the root total): min over lo <= a of S(lo, b), smallest lo on ties
    int a, b;
    {
        const int plo = act ? t.plo[v] : -1, phi = act ? t.phi[v] : -1;
        if (root) { a = plo >= 0 ? plo : LT - 1; b = plo >= 0 ? phi : 0; }
        else { a = gl; b = gl; if (plo >= 0) { a = min(a, plo); b = max(b, phi); } }
    }
    uint32_t B = FGR_INF;
    int blo = 0;
    {
        const uint32_t* sc = t.S + b;
#pragma unroll
        for (int lo = 0; lo < LT; lo++) {
            const uint32_t sv = sc[lo * ES];
            if (lo <= a && sv < B) { B = sv; blo = lo; }
        }
    }
    const uint32_t sbyte = ((uint32_t)blo << 4) | t.HA[blo * ES + b];
    if (root && act && gl == 0) { t.span[0] = (uint8_t)sbyte; *rootcost = B; }
    act = act && !root;
    // edge v -> parent
    uint32_t legA = 0, legB = 0;
    bool straight = false;
    int edir = 0;
    if (act) {
        legA = t.LA[v * ES + gl];
        legB = t.LB[v * ES + gl];
        const int u = t.par[v];
        const bool sh = t.y[v] == t.y[u];
        straight = sh || t.x[v] == t.x[u];
        edir = sh ? 0 : 1;
        t.BW[gl] = B;
        t.BW[ES + gl] = sat_add(B, legA);
    }
    __syncwarp();
    if (act) {
        uint32_t best = FGR_INF;
        int bls = gl;
        if (hm) {                 // hybrid edge: E_v(lt) = min_ls [B_v(ls) + M_e(ls, lt)]
            const uint4* bp = reinterpret_cast<const uint4*>(t.BW);
            uint32_t bs[ES];
#pragma unroll
            for (int q = 0; q < ES / 4; q++) {
                const uint4 w = bp[q];
                bs[4 * q] = w.x; bs[4 * q + 1] = w.y; bs[4 * q + 2] = w.z; bs[4 * q + 3] = w.w;
            }
#pragma unroll
            for (int ls = 0; ls < LT; ls++) {
                const uint32_t cst = sat_add(bs[ls], hm[ls]);
                if (cst < best) { best = cst; bls = ls; }
            }
        } else if (straight) {    // one leg, ls = lt (R7)
            if (c.my_dir == edir) best = sat_add(B, legA);
        } else {
            const uint4* wp = reinterpret_cast<const uint4*>(t.BW + ES);
            uint32_t w1[ES];
#pragma unroll
            for (int q = 0; q < ES / 4; q++) {
                const uint4 w = wp[q];
                w1[4 * q] = w.x; w1[4 * q + 1] = w.y; w1[4 * q + 2] = w.z; w1[4 * q + 3] = w.w;
            }
#pragma unroll
            for (int ls = 0; ls < LT; ls++) {
                const uint32_t cst = sat_add(w1[ls], c.vmeo[ls]);
                if (cst < best) { best = cst; bls = ls; }
            }
            best = sat_add(best, legB);
        }
        t.E[v * ES + gl] = best;
        t.recE[v * ES + gl] = (uint8_t)bls;
        t.recB[v * ES + gl] = (uint8_t)sbyte;
    }
    __syncwarp();
}

// Leg gathers: task = (node i >= 1, line type, quad q of the line's slots).  Type 0: H row
// y_v -> LA, 1: H row y_u -> LB, 2: V column x_v -> LA, 3: V column x_u -> LB.  A quad
// reads 16 B of P and of SB at both ends of the leg (prefix difference, exact in uint32).
struct GTask {
    const uint4* pa;
    const uint4* pb;
    const uint4* sa;
    const uint4* sb;
    uint32_t* dst;     // LA or LB row of node i
    const uint8_t* los;
    int s0, cnt;       // first slot of the quad, slots of the direction
    bool on;
};

__device__ __forceinline__ GTask wtask(const GridView& g, const WHdr* wh, const WTabs& t, int ES, int i, int r,
                                       int qh_shift, int qv_shift) {
    const int nqH = 1 << qh_shift;
    int type, q;
    if (r < 2 * nqH) { type = r >> qh_shift; q = r & (nqH - 1); }
    else { r -= 2 * nqH; type = 2 + (r >> qv_shift); q = r & ((1 << qv_shift) - 1); }
    GTask k;
    const int u = t.par[i];
    const int xv = t.x[i], yv = t.y[i], xu = t.x[u], yu = t.y[u];
    const bool sh = (yv == yu), sv = (xv == xu);
    k.on = !((sh && type != 0) || (sv && type != 2));
    const DirView& d = type < 2 ? g.h : g.v;
    const int line = type == 0 ? yv : type == 1 ? yu : type == 2 ? xv : xu;
    const int a = type < 2 ? min(xv, xu) : min(yv, yu), b = type < 2 ? max(xv, xu) : max(yv, yu);
    const size_t lb = (size_t)line * d.len, sb = (size_t)line * d.nseg;
    k.pa = reinterpret_cast<const uint4*>(d.P + (lb + a) * d.W) + q;
    k.pb = reinterpret_cast<const uint4*>(d.P + (lb + b) * d.W) + q;
    k.sa = reinterpret_cast<const uint4*>(d.SB + (sb + (a >> FGR_SEG_SHIFT)) * d.W) + q;
    k.sb = reinterpret_cast<const uint4*>(d.SB + (sb + (b >> FGR_SEG_SHIFT)) * d.W) + q;
    k.dst = ((type & 1) ? t.LB : t.LA) + i * ES;
    k.los = wh->los[type < 2 ? 0 : 1];
    k.s0 = 4 * q;
    k.cnt = d.cnt;
    return k;
}

template <int LT, int MC, int WARPS>
__global__ void __launch_bounds__(32 * WARPS, MC <= 8 ? 5 : 4) k_dp_walk(GridView g, NetsView nv, const int32_t* __restrict__ list,
                                                         int count, Out o, int commit, HybView hy) {
    constexpr int G = WK<LT>::G, ES = WK<LT>::ES;
    extern __shared__ __align__(16) unsigned char smem[];
    WHdr* wh = reinterpret_cast<WHdr*>(smem);
    init_hdr(&wh->h, g);
    for (int i = threadIdx.x; i < 2 * FGR_MAXL; i += blockDim.x) wh->los[i / FGR_MAXL][i % FGR_MAXL] = g.layer_of_slot[i / FGR_MAXL][i % FGR_MAXL];
    __syncthreads();
    const Hdr* h = &wh->h;
    const int warp = threadIdx.x >> 5, lane = lane_id();
    const int idx0 = (blockIdx.x * WARPS + warp) * G;
    if (idx0 >= count) return;
    const int gi = lane / LT < G ? lane / LT : G;   // my group (G = idle lane)
    const int gl = lane - gi * LT;                  // my layer inside the group
    const bool glane = gi < G;
    const size_t TB = wtabs_bytes(MC, LT);
    unsigned char* wbase = smem + a16(sizeof(WHdr)) + (size_t)warp * G * TB;
    auto tabs_of = [&](int q) { return carve_w(wbase + (size_t)q * TB, MC, LT); };
    WLane<LT> c;
    c.load(h, gl);
    int net_l = -1, a0_l = 0, m_l = 0, hn_l = -1;
    if (lane < G && idx0 + lane < count) {
        net_l = list[idx0 + lane];
        a0_l = nv.off[net_l];
        m_l = nv.off[net_l + 1] - a0_l;
        if (hy.net) hn_l = hy.net[net_l];
    }
    int mq[G], aq[G];
#pragma unroll
    for (int q = 0; q < G; q++) { mq[q] = __shfl_sync(0xffffffffu, m_l, q); aq[q] = __shfl_sync(0xffffffffu, a0_l, q); }
    int my_m = 0, my_a = 0, my_hn = -1;
#pragma unroll
    for (int q = 0; q < G; q++) {
        const int hq = __shfl_sync(0xffffffffu, hn_l, q);
        my_m = (gi == q) ? mq[q] : my_m;
        my_a = (gi == q) ? aq[q] : my_a;
        my_hn = (gi == q) ? hq : my_hn;
    }
    Flat<G> nodes;
    nodes.build(mq);
    for (int it = lane; it < nodes.total(); it += 32) {
        const int q = nodes.group(it), i = it - nodes.base(q);
        int a = 0;
#pragma unroll
        for (int k = 0; k < G; k++) a = (k == q) ? aq[k] : a;
        const WTabs t = tabs_of(q);
        t.x[i] = nv.x[a + i]; t.y[i] = nv.y[a + i]; t.par[i] = (uint16_t)nv.par[a + i];
        t.plo[i] = nv.plo[a + i]; t.phi[i] = nv.phi[a + i];
        t.cm[i] = 0;
    }
    __syncwarp();
    for (int it = lane; it < nodes.total(); it += 32) {
        const int q = nodes.group(it), i = it - nodes.base(q);
        if (i > 0) { const WTabs t = tabs_of(q); atomicOr(&t.cm[t.par[i]], 1u << i); }
    }
    // all leg gathers of the G nets, NF tasks per lane in flight
    constexpr int NF = MC <= 8 ? 2 : 4;
    const int qh_shift = g.h.W == 4 ? 0 : (g.h.W == 8 ? 1 : 2), qv_shift = g.v.W == 4 ? 0 : (g.v.W == 8 ? 1 : 2);
    const int tpe_shift_h = qh_shift + 1;
    const int TPE = (2 << qh_shift) + (2 << qv_shift);   // tasks per edge
    (void)tpe_shift_h;
    int tq[G];
#pragma unroll
    for (int q = 0; q < G; q++) tq[q] = mq[q] > 1 ? TPE * (mq[q] - 1) : 0;
    Flat<G> tasks;
    tasks.build(tq);
    for (int it0 = lane; it0 < tasks.total(); it0 += NF * 32) {
        GTask k[NF];
        uint4 r[NF][4];
#pragma unroll
        for (int j = 0; j < NF; j++) {
            const int it = it0 + 32 * j;
            k[j].on = false;
            if (it < tasks.total()) {
                const int q = tasks.group(it), ti = it - tasks.base(q);
                const int i = 1 + ti / TPE;
                k[j] = wtask(g, wh, tabs_of(q), ES, i, ti - (i - 1) * TPE, qh_shift, qv_shift);
                if (k[j].on) {
                    r[j][0] = __ldg(k[j].pa); r[j][1] = __ldg(k[j].pb);
                    if (k[j].sa != k[j].sb) { r[j][2] = __ldg(k[j].sa); r[j][3] = __ldg(k[j].sb); }
                    else { r[j][2] = make_uint4(0, 0, 0, 0); r[j][3] = r[j][2]; }   // one segment: bases cancel
                }
            }
        }
#pragma unroll
        for (int j = 0; j < NF; j++) {
            if (k[j].on) {
                const uint32_t d[4] = {(r[j][3].x + r[j][1].x) - (r[j][2].x + r[j][0].x),
                                       (r[j][3].y + r[j][1].y) - (r[j][2].y + r[j][0].y),
                                       (r[j][3].z + r[j][1].z) - (r[j][2].z + r[j][0].z),
                                       (r[j][3].w + r[j][1].w) - (r[j][2].w + r[j][0].w)};
#pragma unroll
                for (int s = 0; s < 4; s++)
                    if (k[j].s0 + s < k[j].cnt) k[j].dst[k[j].los[k[j].s0 + s]] = d[s];
            }
        }
    }
    __syncwarp();
    // bottom-up DP: descending node index is children-first (parent[i] < i)
    int maxm = 0;
#pragma unroll
    for (int q = 0; q < G; q++) maxm = max(maxm, mq[q]);
    const WTabs t = tabs_of(glane ? gi : 0);
    for (int k = 0; k + 1 < maxm; k++) {
        const int v = my_m - 1 - k;
        const bool act = glane && v >= 1;
        const uint32_t* hm = nullptr;   // hybrid edge: its transfer matrix column for lt = gl
        if (act && my_hn >= 0) {
            const int hs = hy.slot[my_a + v];
            if (hs >= 0) hm = hy.M + ((size_t)hs * LT + gl) * LT;
        }
        wstep<LT, false>(c, t, v, act, false, gl, hm, nullptr);
    }
    __shared__ uint32_t s_cost[WARPS * 4];
    wstep<LT, false>(c, t, 0, glane && my_m >= 2, true, gl, nullptr, &s_cost[warp * 4 + (glane ? gi : 0)]);
    __syncwarp();
    // S5: one lane per net walks the nodes in ascending index (parents first)
    if (glane && gl == 0) {
        for (int v = 1; v < my_m; v++) {
            const int u = t.par[v];
            const int sp = t.span[u];
            const int lo = sp >> 4, hi = sp & 15;
            const uint4* ep = reinterpret_cast<const uint4*>(t.E + v * ES);
            uint32_t e[ES];
#pragma unroll
            for (int q = 0; q < ES / 4; q++) {
                const uint4 w = ep[q];
                e[4 * q] = w.x; e[4 * q + 1] = w.y; e[4 * q + 2] = w.z; e[4 * q + 3] = w.w;
            }
            uint32_t be = 0xFFFFFFFFu;
            int lt = lo;
#pragma unroll
            for (int l = 0; l < LT; l++)
                if (l >= lo && l <= hi && e[l] < be) { be = e[l]; lt = l; }   // smallest l attaining the min (R11)
            const int ls = t.recE[v * ES + lt];
            t.span[v] = t.recB[v * ES + ls];
            const bool straight = (t.x[v] == t.x[u]) || (t.y[v] == t.y[u]);
            const uint32_t bend = seg_bend(h->dir[ls], h->dir[lt], straight);
            t.seg[v] = bend | ((uint32_t)ls << 8) | ((uint32_t)lt << 16) | ((uint32_t)straight << 24);
        }
    }
    __syncwarp();
    // outputs and S6
    for (int it = lane; it < nodes.total(); it += 32) {
        const int q = nodes.group(it), i = it - nodes.base(q);
        const WTabs tt = tabs_of(q);
        const uint32_t s = i ? tt.seg[i] : 0xFFFFFFFFu;
        int a = 0;
#pragma unroll
        for (int k = 0; k < G; k++) a = (k == q) ? aq[k] : a;
        if (o.rec_seg) o.rec_seg[o.rec_off[o.list_base + idx0 + q] + i] = s;
        else o.seg[a + i] = s;
        if (commit && i > 0) {
            const int u = tt.par[i];
            commit_edge(g, h, tt.x[i], tt.y[i], tt.x[u], tt.y[u], s, hyb_z(hy, a + i, s, LT));
        }
    }
    if (glane && gl == 0 && my_m >= 1) {
        const uint32_t total = my_m >= 2 ? s_cost[warp * 4 + gi] : 0u;
        if (o.rec_seg) o.rec_cost[o.list_base + idx0 + gi] = total;
        else o.cost[list[idx0 + gi]] = total;
    }
}


// ------------------------------------------------------------- large nets (> 32 nodes)
// One CTA per net, the same node step as a dataflow over the tree: lane groups take the
// leaves by ticket and walk upwards; a group that finishes node v decrements the pending
// child count of v's parent and continues with the parent when it was the last child
// (no level barriers, no waiting: the tree is a DAG of one-way hand-offs).  Values are
// exact whatever the order (saturating integer sums and minima commute), so the result is
// the oracle's.  Backtrack: one thread per node in ascending index, waiting on its
// parent's span flag (parents first, R22).
constexpr int kRing = 24;        // root-path transfer matrices in flight (ring slots)
constexpr int kWalkerMin = 64;   // root paths at least this long get the walker warp

__host__ __device__ inline size_t flow_bytes(int m, int L, int warps) {
    const size_t ES = (size_t)((L + 3) & ~3);
    const size_t scratch = a16(L * ES * 4) + a16(L * ES) + a16(2 * ES * 4);
    return wtabs_bytes(m, L) + a16((size_t)(m + 1) * 2) + 6 * a16((size_t)m * 2) + a16((size_t)m) +
           (size_t)kRing * L * ES * 4 + (size_t)warps * groups_of(L) * scratch;
}


// Value-only transfer matrix of a root-path node v with heavy child h (the product form of
// the node and edge steps; exact because saturating min-plus is associative and distributes):
//   E_v(lt) = min_l [E_h(l) + M_v(l, lt)],  M_v(l, lt) = min_ls [G_v(hull(l, ls, pins)) + W_v(ls, lt)],
// G_v(a, b) = min over spans [lo, hi] with lo <= a, hi >= b of V(lo, hi) + sum_{light c} min_{[lo,hi]} E_c,
// W_v = the edge step (legs + bend via, or the hybrid matrix).  Lane lt writes mrow[lt * ES + l].
template <int LT>
__device__ __forceinline__ void build_tm(const WLane<LT>& c, const WTabs& t, int v, int heavy, bool act, int gl,
                                         const uint32_t* hm, const uint16_t* cs, const uint16_t* cl, uint32_t* mrow) {
    constexpr int ES = WK<LT>::ES;
    uint32_t acc[LT];
#pragma unroll
    for (int hi = 0; hi < LT; hi++) acc[hi] = c.vrow[hi];
    int ck = act ? cs[v] : 0;
    const int ce = act ? cs[v + 1] : 0;
    for (; ck < ce; ck++) {
        const int ch = cl[ck];
        if (ch == heavy) continue;
        const uint4* ep = reinterpret_cast<const uint4*>(t.E + ch * ES);
        uint32_t e[ES];
#pragma unroll
        for (int q = 0; q < ES / 4; q++) {
            const uint4 w = ep[q];
            e[4 * q] = w.x; e[4 * q + 1] = w.y; e[4 * q + 2] = w.z; e[4 * q + 3] = w.w;
        }
        uint32_t run = FGR_INF;
#pragma unroll
        for (int hi = 0; hi < LT; hi++) {
            run = min(run, hi >= gl ? e[hi] : FGR_INF);
            acc[hi] = sat_add(acc[hi], run);
        }
    }
    if (act) {   // suffix minima over hi (values only)
        uint32_t srow[ES];
#pragma unroll
        for (int hi = LT; hi < ES; hi++) srow[hi] = FGR_INF;
        uint32_t sm = FGR_INF;
#pragma unroll
        for (int hi = LT - 1; hi >= 0; hi--) { sm = min(sm, acc[hi]); srow[hi] = sm; }
        uint4* sp = reinterpret_cast<uint4*>(t.S + gl * ES);
#pragma unroll
        for (int q = 0; q < ES / 4; q++) sp[q] = make_uint4(srow[4 * q], srow[4 * q + 1], srow[4 * q + 2], srow[4 * q + 3]);
    }
    __syncwarp();
    if (act) {   // G(a, b) = min_{lo <= a} S(lo, b): lane b owns column b
        uint32_t run = FGR_INF;
#pragma unroll
        for (int a = 0; a < LT; a++) { run = min(run, t.S[a * ES + gl]); t.S[a * ES + gl] = run; }
    }
    __syncwarp();
    if (act) {
        const int u = t.par[v];
        const bool sh = t.y[v] == t.y[u];
        const bool straight = sh || t.x[v] == t.x[u];
        const int edir = sh ? 0 : 1;
        const uint32_t legB = t.LB[v * ES + gl];
        uint32_t w[LT];
#pragma unroll
        for (int ls = 0; ls < LT; ls++) {
            if (hm) w[ls] = hm[ls];
            else if (straight) w[ls] = (ls == gl && c.my_dir == edir) ? t.LA[v * ES + gl] : FGR_INF;
            else w[ls] = sat_add(sat_add(t.LA[v * ES + ls], c.vmeo[ls]), legB);
        }
        const int plo = t.plo[v], phi = t.phi[v];
        uint32_t col[ES];
#pragma unroll
        for (int l = LT; l < ES; l++) col[l] = FGR_INF;
#pragma unroll
        for (int l = 0; l < LT; l++) {
            uint32_t best = FGR_INF;
#pragma unroll
            for (int ls = 0; ls < LT; ls++) {
                int lo = min(l, ls), hi = max(l, ls);
                if (plo >= 0) { lo = min(lo, plo); hi = max(hi, phi); }
                best = min(best, sat_add(t.S[lo * ES + hi], w[ls]));
            }
            col[l] = best;
        }
        uint4* mp = reinterpret_cast<uint4*>(mrow + gl * ES);
#pragma unroll
        for (int q = 0; q < ES / 4; q++) mp[q] = make_uint4(col[4 * q], col[4 * q + 1], col[4 * q + 2], col[4 * q + 3]);
    }
    __syncwarp();
}

// Root-path state packed above the pending-children count of a node: atomicSub on the
// count leaves it alone.  0 pending, 1 building, 2 matrix ready, 3 walker inline, 4 kicked.
#define FST(w) ((w) >> 16)
#define FCNT(w) ((w) & 0xFFFFu)

template <int LT, int WARPS>
__global__ void __launch_bounds__(32 * WARPS) k_dp_flow(GridView g, NetsView nv, const int32_t* __restrict__ list,
                                                         int count, Out o, int commit, Prep prep, HybView hy) {
    constexpr int G = WK<LT>::G, ES = WK<LT>::ES;
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ int s_ticket, s_nleaf, s_ticket2, s_ntops, s_K, s_wpos, s_wdone, s_kqh, s_kqt;
#ifdef FGR_TIMING
    __shared__ long long s_wst[4];   // walker: fast steps, inline steps, cycles waiting for a state, cycles waiting for light children
    if (threadIdx.x < 4) s_wst[threadIdx.x] = 0;
#endif
    __shared__ uint32_t s_cost;
    WHdr* wh = reinterpret_cast<WHdr*>(smem);
    init_hdr(&wh->h, g);
    for (int i = threadIdx.x; i < 2 * FGR_MAXL; i += blockDim.x) wh->los[i / FGR_MAXL][i % FGR_MAXL] = g.layer_of_slot[i / FGR_MAXL][i % FGR_MAXL];
    const int tid = threadIdx.x, T = blockDim.x, warp = tid >> 5, lane = lane_id();
#ifdef FGR_TIMING
    long long tm[6];
    tm[0] = clock64();
#define FMARK(i) do { tm[i] = clock64(); } while (0)
#else
#define FMARK(i) do { } while (0)
#endif
    if (tid == 0) { s_ticket = 0; s_nleaf = 0; s_cost = 0; s_ticket2 = 0; s_ntops = 0; s_wpos = 0; s_wdone = 0; s_kqh = 0; s_kqt = 0; }
    const int net = list[blockIdx.x];
    const int a0 = nv.off[net], m = nv.off[net + 1] - a0;
    const int hnet = hy.net ? hy.net[net] : -1;
    unsigned char* p = smem + a16(sizeof(WHdr));
    const WTabs t = carve_w(p, m, LT);
    p += wtabs_bytes(m, LT);
    uint16_t* cs = (uint16_t*)p; p += a16((size_t)(m + 1) * 2);
    uint16_t* cl = (uint16_t*)p; p += a16((size_t)m * 2);
    uint16_t* leafq = (uint16_t*)p; p += a16((size_t)m * 2);
    uint16_t* hv = (uint16_t*)p; p += a16((size_t)m * 2);     // heavy child (backtrack paths), 0xFFFF at a leaf
    uint16_t* rpos = (uint16_t*)p; p += a16((size_t)m * 2);   // index along the root path from its bottom, 0xFFFF off
    uint16_t* rp = (uint16_t*)p; p += a16((size_t)m * 2);     // root path, bottom first
    uint16_t* kq = (uint16_t*)p; p += a16((size_t)m * 2);     // kicked matrix builds (walker -> workers)
    uint32_t* mslots = (uint32_t*)p; p += (size_t)kRing * LT * ES * 4;
    uint8_t* sready = p; p += a16((size_t)m);
    unsigned char* scr = p;
    __syncthreads();
    for (int i = tid; i < m; i += T) {
        t.x[i] = nv.x[a0 + i]; t.y[i] = nv.y[a0 + i]; t.par[i] = (uint16_t)nv.par[a0 + i];
        t.plo[i] = nv.plo[a0 + i]; t.phi[i] = nv.phi[a0 + i];
        sready[i] = 0;
        t.cm[i] = 0;
    }
    if (prep.cs) {   // child CSR from the once-per-stage tree analysis
        for (int i = tid; i < m; i += T) { cs[i] = prep.cs[a0 + i]; cl[i] = prep.cl[a0 + i]; }
        if (tid == 0) cs[m] = (uint16_t)(m - 1);
        __syncthreads();
    } else {         // build it here: counts, one warp's exclusive scan, fill
        __syncthreads();
        for (int i = 1 + tid; i < m; i += T) atomicAdd(&t.cm[t.par[i]], 1u);
        __syncthreads();
        if (warp == 0) {
            uint32_t carry = 0;
            for (int c0 = 0; c0 < m; c0 += 32) {
                const int i = c0 + lane;
                const uint32_t v = i < m ? t.cm[i] : 0u;
                uint32_t inc = v;
#pragma unroll
                for (int off = 1; off < 32; off <<= 1) {
                    const uint32_t q = __shfl_up_sync(0xffffffffu, inc, off);
                    if (lane >= off) inc += q;
                }
                if (i < m) { cs[i] = (uint16_t)(carry + inc - v); t.seg[i] = carry + inc - v; }
                carry += __shfl_sync(0xffffffffu, inc, 31);
            }
            if (lane == 0) cs[m] = (uint16_t)carry;
        }
        __syncthreads();
        for (int i = 1 + tid; i < m; i += T) cl[atomicAdd(&t.seg[t.par[i]], 1u)] = (uint16_t)i;
        __syncthreads();
    }
    for (int i = tid; i < m; i += T) {
        const uint32_t nc = (uint32_t)(cs[i + 1] - cs[i]);
        hv[i] = prep.hv ? prep.hv[a0 + i] : (nc ? cl[cs[i]] : (uint16_t)0xFFFF);
        rpos[i] = prep.rpos ? prep.rpos[a0 + i] : (uint16_t)0xFFFF;
    }
    __syncthreads();
    if (!prep.rpos && tid == 0) {   // root path = the heavy chain from the root
        int k = 0;
        for (int w = 0; w != 0xFFFF; w = hv[w]) k++;
        int j = k - 1;
        for (int w = 0; w != 0xFFFF; w = hv[w]) rpos[w] = (uint16_t)(j--);
    }
    __syncthreads();
    for (int i = tid; i < m; i += T) if (rpos[i] != 0xFFFF) rp[rpos[i]] = (uint16_t)i;
    if (tid == 0) s_K = rpos[0] + 1;
    __syncthreads();
    const int K = s_K;
    const bool usew = K >= kWalkerMin;   // a root-path walker pays off only on long chains
    // pending children: all of them off the root path, the light ones on it (the walker owns
    // the heavy chain).  Work queue: matrix builds of the first root-path nodes without light
    // children, then the leaves off the root path.
    if (tid == 0) {
        int n = 0;
        for (int k = 1; usew && k < K - 1 && k < kRing; k++) {
            const int v = rp[k];
            if (cs[v + 1] - cs[v] == 1) leafq[n++] = (uint16_t)(v | 0x8000);
        }
        s_nleaf = n;
    }
    __syncthreads();
    for (int i = tid; i < m; i += T) {
        const uint32_t nc = (uint32_t)(cs[i + 1] - cs[i]);
        const bool onrp = usew && rpos[i] != 0xFFFF;
        t.cm[i] = onrp ? (nc ? nc - 1 : 0) : nc;
        if (nc == 0 && !onrp) leafq[atomicAdd(&s_nleaf, 1)] = (uint16_t)i;
    }
    FMARK(1);
    pdl_wait();   // the refresh that precedes this launch must be done before the gathers
    {
        constexpr int NF = 4;
        const int qh_shift = g.h.W == 4 ? 0 : (g.h.W == 8 ? 1 : 2), qv_shift = g.v.W == 4 ? 0 : (g.v.W == 8 ? 1 : 2);
        const int TPE = (2 << qh_shift) + (2 << qv_shift);
        const int total = TPE * (m - 1);
        for (int it0 = tid; it0 < total; it0 += NF * T) {
            GTask k[NF];
            uint4 r[NF][4];
#pragma unroll
            for (int j = 0; j < NF; j++) {
                const int it = it0 + T * j;
                k[j].on = false;
                if (it < total) {
                    const int i = 1 + it / TPE;
                    k[j] = wtask(g, wh, t, ES, i, it - (i - 1) * TPE, qh_shift, qv_shift);
                    if (k[j].on) {
                        r[j][0] = __ldg(k[j].pa); r[j][1] = __ldg(k[j].pb);
                        if (k[j].sa != k[j].sb) { r[j][2] = __ldg(k[j].sa); r[j][3] = __ldg(k[j].sb); }
                        else { r[j][2] = make_uint4(0, 0, 0, 0); r[j][3] = r[j][2]; }   // one segment: bases cancel
                    }
                }
            }
#pragma unroll
            for (int j = 0; j < NF; j++) {
                if (k[j].on) {
                    const uint32_t d[4] = {(r[j][3].x + r[j][1].x) - (r[j][2].x + r[j][0].x),
                                           (r[j][3].y + r[j][1].y) - (r[j][2].y + r[j][0].y),
                                           (r[j][3].z + r[j][1].z) - (r[j][2].z + r[j][0].z),
                                           (r[j][3].w + r[j][1].w) - (r[j][2].w + r[j][0].w)};
#pragma unroll
                    for (int s2 = 0; s2 < 4; s2++)
                        if (k[j].s0 + s2 < k[j].cnt) k[j].dst[k[j].los[k[j].s0 + s2]] = d[s2];
                }
            }
        }
    }
    __syncthreads();
    FMARK(2);
    const int nleaf = s_nleaf;
    // ---- bottom-up: warp 0 walks the root path with one vector x matrix step per node
    // (M_v built ahead by the workers, else an inline node step); warps 1.. run the
    // dataflow over the rest of the tree and build the root-path matrices as soon as a
    // node's light children are final.
    {
        const int gi = lane / LT < G ? lane / LT : G;
        const int gl = lane - gi * LT;
        const bool glane = gi < G;
        const int gbase = (glane ? gi : 0) * LT;
        const unsigned gmask = glane ? (((1u << LT) - 1u) << gbase) : 0u;
        WTabs tg = t;
        {
            const size_t sz = a16(LT * ES * 4) + a16(LT * ES) + a16(2 * ES * 4);
            unsigned char* q = scr + (size_t)(warp * G + (glane ? gi : 0)) * sz;
            tg.S = (uint32_t*)q; q += a16(LT * ES * 4);
            tg.HA = q; q += a16(LT * ES);
            tg.BW = (uint32_t*)q;
        }
        WLane<LT> c;
        c.load(&wh->h, gl);
        auto hmat = [&](int v) -> const uint32_t* {
            if (hnet < 0 || v <= 0) return nullptr;
            const int hs = hy.slot[a0 + v];
            return hs >= 0 ? hy.M + ((size_t)hs * LT + gl) * LT : nullptr;
        };
        // matrix build of root-path node v (index k) by a lane group that claimed it
        auto build = [&](int v, int k, bool act) {
            build_tm<LT>(c, tg, v, hv[v], act, gl, act ? hmat(v) : nullptr, cs, cl, mslots + (size_t)(k % kRing) * LT * ES);
            if (act) __threadfence_block();
            __syncwarp();
            if (act && gl == 0) atomicAdd(&t.cm[v], (2u - 1u) << 16);   // state 1 -> 2
        };
        // claim the build of root-path node v (k = rpos): state 0 -> 1 if its ring slot is free
        auto claim = [&](int v, int k, uint32_t from) -> bool {
            if (k >= *(volatile int*)&s_wpos + kRing) return false;
            const uint32_t w = *(volatile uint32_t*)&t.cm[v];
            if (FST(w) != from || FCNT(w) != 0) return false;
            return atomicCAS(&t.cm[v], w, (1u << 16)) == w;
        };
        if (usew && warp == 0) {
            const bool act = gi == 0;   // one lane group walks; the warp's other lanes idle
            uint32_t Eprev = 0;
            (void)Eprev;
            for (int k = 0; k < K; k++) {
                const int v = rp[k];
                if (k == 0) {            // bottom leaf
                    wstep<LT, true>(c, tg, v, act, false, gl, act ? hmat(v) : nullptr, &s_cost, cs, cl);
                } else if (k == K - 1) { // the root: wait for its light children, generalised Eq. (4)
                    while (FCNT(*(volatile uint32_t*)&t.cm[0]) != 0) __nanosleep(20);
                    __threadfence_block();
                    wstep<LT, true>(c, tg, 0, act, true, gl, nullptr, &s_cost, cs, cl);
                } else {
                    bool fast = false;
#ifdef FGR_TIMING
                    const long long tw0 = clock64();
#endif
                    for (;;) {
                        uint32_t w = *(volatile uint32_t*)&t.cm[v];
                        const uint32_t st = FST(w);
                        if (st == 2) { fast = true; break; }
                        if (st == 0 || st == 4) {
                            uint32_t old = 0;
                            if (lane == 0) old = atomicCAS(&t.cm[v], w, (w & 0xFFFFu) | (3u << 16));
                            old = __shfl_sync(0xffffffffu, old, 0);
                            if (old == w) break;   // inline
                        }
                        // st == 1: a worker is building it
                    }
                    __threadfence_block();
#ifdef FGR_TIMING
                    if (lane == 0) { s_wst[fast ? 0 : 1]++; s_wst[2] += clock64() - tw0; }
#endif
                    if (fast) {
                        if (act) {
                            const uint4* ep = reinterpret_cast<const uint4*>(t.E + rp[k - 1] * ES);
                            const uint4* mp = reinterpret_cast<const uint4*>(mslots + (size_t)(k % kRing) * LT * ES + gl * ES);
                            uint32_t e[ES], mc[ES];
#pragma unroll
                            for (int q = 0; q < ES / 4; q++) {
                                const uint4 a = ep[q], b = mp[q];
                                e[4 * q] = a.x; e[4 * q + 1] = a.y; e[4 * q + 2] = a.z; e[4 * q + 3] = a.w;
                                mc[4 * q] = b.x; mc[4 * q + 1] = b.y; mc[4 * q + 2] = b.z; mc[4 * q + 3] = b.w;
                            }
                            uint32_t best = FGR_INF;
#pragma unroll
                            for (int l = 0; l < LT; l++) best = __viaddmin_u32(e[l], mc[l], best);   // e + m <= 2^32 - 2
                            t.E[v * ES + gl] = best;
                        }
                        __syncwarp();
                    } else {
#ifdef FGR_TIMING
                        const long long tw1 = clock64();
#endif
                        while (FCNT(*(volatile uint32_t*)&t.cm[v]) != 0) __nanosleep(20);
                        __threadfence_block();
#ifdef FGR_TIMING
                        if (lane == 0) s_wst[3] += clock64() - tw1;
#endif
                        wstep<LT, true>(c, tg, v, act, false, gl, act ? hmat(v) : nullptr, &s_cost, cs, cl);
                    }
                }
                __threadfence_block();
                __syncwarp();
                if (lane == 0) {
                    *(volatile int*)&s_wpos = k + 1;
                    // the ring slot of k + kRing is free now: kick its build if it was skipped
                    const int kk = k + kRing;
                    if (kk < K - 1) {
                        const int vk = rp[kk];
                        const uint32_t w = *(volatile uint32_t*)&t.cm[vk];
                        if (FST(w) == 0 && FCNT(w) == 0 && atomicCAS(&t.cm[vk], w, 4u << 16) == w) {
                            const int tpos = s_kqt;
                            kq[tpos] = (uint16_t)vk;
                            __threadfence_block();
                            *(volatile int*)&s_kqt = tpos + 1;
                        }
                    }
                }
            }
            if (lane == 0) { __threadfence_block(); *(volatile int*)&s_wdone = 1; }
        } else {
            int cur = -1;          // node to step (walk), or 0x8000 | v for a matrix build
            bool more = true;      // queue not exhausted (leader's view)
            bool fin = false;      // no work will come to this group any more
            for (;;) {
                if (glane && cur < 0 && !fin) {
                    // never wait here: a group of this warp may hold a node the walker needs
                    int tk = -1, f = 0;
                    if (gl == 0) {
                        const int h = *(volatile int*)&s_kqh;
                        if (h < *(volatile int*)&s_kqt) {   // kicked builds first
                            if (atomicCAS(&s_kqh, h, h + 1) == h) { __threadfence_block(); tk = 0x10000 | kq[h]; }
                        } else if (more) {
                            const int q = atomicAdd(&s_ticket, 1);
                            if (q < nleaf) tk = leafq[q];
                            else more = false;
                        } else if ((!usew || *(volatile int*)&s_wdone) && h >= *(volatile int*)&s_kqt) {
                            f = 1;
                        }
                    }
                    tk = __shfl_sync(gmask, tk, gbase);
                    fin = __shfl_sync(gmask, f, gbase) != 0;
                    if (tk >= 0x10000) {   // kicked: state 4 -> 1
                        const int v = tk & 0xFFFF;
                        uint32_t ok = 0;
                        if (gl == 0) ok = atomicCAS(&t.cm[v], 4u << 16, 1u << 16) == (4u << 16);
                        ok = __shfl_sync(gmask, ok, gbase);
                        cur = ok ? (0x8000 | v) : -1;
                    } else if (tk >= 0 && (tk & 0x8000)) {   // queued build: state 0 -> 1
                        const int v = tk & 0x7FFF;
                        uint32_t ok = 0;
                        if (gl == 0) ok = claim(v, rpos[v], 0) ? 1u : 0u;
                        ok = __shfl_sync(gmask, ok, gbase);
                        cur = ok ? tk : -1;
                    } else {
                        cur = tk;
                    }
                }
                const bool busy = glane && cur >= 0;
                if (!__any_sync(0xffffffffu, glane && !fin)) break;
                if (!__any_sync(0xffffffffu, busy)) { __nanosleep(100); continue; }
                const bool bld = busy && (cur & 0x8000);
                const int v = busy ? (cur & 0x7FFF) : 0;
                // the warp's groups may mix builds and node steps: both calls run warp-wide
                build(v, bld ? rpos[v] : 0, bld);
                const bool stp = busy && !bld;
                wstep<LT, true>(c, tg, stp ? v : 0, stp, stp && v == 0, gl, stp ? hmat(v) : nullptr, &s_cost, cs, cl);
                if (busy) __threadfence_block();
                __syncwarp();
                if (busy) {
                    int nxt = -1;
                    if (gl == 0 && stp && v != 0) {
                        const int pu = t.par[v];
                        if (FCNT(atomicSub(&t.cm[pu], 1u)) == 1u) {   // last child
                            if (!usew || rpos[pu] == 0xFFFF) nxt = pu;  // continue up
                            else if (pu != 0 && claim(pu, rpos[pu], 0)) nxt = 0x8000 | pu;   // build its matrix
                        }
                    }
                    nxt = __shfl_sync(gmask, nxt, gbase);
                    __threadfence_block();
                    cur = nxt;
                }
            }
        }
    }
    __syncthreads();
    // recE / recB of the root-path nodes the walker passed with a matrix step: independent
    // node steps now that every E is final (same E values, R11 argmins)
    {
        const int gi = lane / LT < G ? lane / LT : G;
        const int gl = lane - gi * LT;
        const bool glane = gi < G;
        const int gbase = (glane ? gi : 0) * LT;
        const unsigned gmask = glane ? (((1u << LT) - 1u) << gbase) : 0u;
        WTabs tg = t;
        {
            const size_t sz = a16(LT * ES * 4) + a16(LT * ES) + a16(2 * ES * 4);
            unsigned char* q = scr + (size_t)(warp * G + (glane ? gi : 0)) * sz;
            tg.S = (uint32_t*)q; q += a16(LT * ES * 4);
            tg.HA = q; q += a16(LT * ES);
            tg.BW = (uint32_t*)q;
        }
        WLane<LT> c;
        c.load(&wh->h, gl);
        if (tid == 0) s_ticket = 0;
        __syncthreads();
        for (; usew;) {
            int k = -1;
            if (glane && gl == 0) {
                for (;;) {
                    const int q = atomicAdd(&s_ticket, 1);
                    if (q >= K - 2) break;
                    if (FST(t.cm[rp[q + 1]]) == 2) { k = q + 1; break; }
                }
            }
            if (glane) k = __shfl_sync(gmask, k, gbase);
            const bool act = glane && k > 0;
            if (!__any_sync(0xffffffffu, act)) break;
            const int v = act ? rp[k] : 0;
            const uint32_t* hm = nullptr;
            if (act && hnet >= 0) {
                const int hs = hy.slot[a0 + v];
                if (hs >= 0) hm = hy.M + ((size_t)hs * LT + gl) * LT;
            }
            wstep<LT, true>(c, tg, v, act, false, gl, hm, &s_cost, cs, cl);
        }
    }
    __syncthreads();
    FMARK(3);
    // ---- S5 along heavy paths (the tree analysis puts the deepest chain on the root path):
    // a path starts at the root or at a light child and follows hv[] down to a leaf.  Lane 0
    // of each warp walks one path at a time (a scalar span -> lt -> ls -> span chain); a
    // path top waits for its parent's span.  Paths are ticketed shallowest top first (the
    // tree analysis order, else ascending index), so an awaited path is always held by a
    // running warp: no deadlock.
    if (warp == 0) {
        int n = 0;
        if (prep.pq) {
            const int np = prep.npaths[net];
            for (int k = lane; k < np; k += 32) leafq[k] = prep.pq[a0 + np - 1 - k];
            n = np;
        } else {
            for (int c0 = 0; c0 < m; c0 += 32) {
                const int v = c0 + lane;
                const bool top = v < m && (v == 0 || hv[t.par[v]] != v);
                const unsigned bal = __ballot_sync(0xffffffffu, top);
                if (top) leafq[n + __popc(bal & ((1u << lane) - 1u))] = (uint16_t)v;
                n += __popc(bal);
            }
        }
        if (lane == 0) { s_ntops = n; sready[0] = 1; }   // the root's span came from the forward pass
    }
    __syncthreads();
    const int ntops = s_ntops;
    if constexpr (LT * (LT + 1) / 2 <= 8 * LT) {
        // The backtrack step of a node is a fixed map from its parent's span to its own
        // (same derivation as k_dp_large): tabulated per node by all threads into the dead
        // leg tables (LA, LB), so a path walk is one shared-memory byte load per node; the
        // segment records are derived from the parent's span in the parallel output pass.
        constexpr int NSP = LT * (LT + 1) / 2;
        constexpr int MSB = (NSP + 3) & ~3;
        uint8_t* smap = reinterpret_cast<uint8_t*>(t.LA);
        auto code = [](int sp) -> int {        // (lo << 4 | hi) -> triangular code
            const int lo = sp >> 4, hi = sp & 15;
            return max(0, min(lo * (2 * LT - lo + 1) / 2 + (hi - lo), NSP - 1));
        };
        for (int v = 1 + tid; v < m; v += T) {
            uint32_t ev[LT], cc[LT];
#pragma unroll
            for (int l = 0; l < LT; l++) {
                ev[l] = t.E[v * ES + l];
                cc[l] = (uint32_t)code(t.recB[v * ES + t.recE[v * ES + l]]);
            }
            uint32_t* out = reinterpret_cast<uint32_t*>(smap + (size_t)v * MSB);
            uint32_t word = 0;
            int idx = 0;
#pragma unroll
            for (int lo = 0; lo < LT; lo++) {
                uint32_t be = ev[lo], c0 = cc[lo];
#pragma unroll
                for (int hi = lo; hi < LT; hi++) {
                    if (hi > lo && ev[hi] < be) { be = ev[hi]; c0 = cc[hi]; }
                    word |= c0 << (8 * (idx & 3));
                    if ((idx & 3) == 3) { out[idx >> 2] = word; word = 0; }
                    idx++;
                }
            }
            if (idx & 3) out[idx >> 2] = word;
        }
        if (tid == 0) t.span[0] = (uint8_t)code(t.span[0]);
        __syncthreads();
        if (lane == 0) {
            for (;;) {
                const int k = atomicAdd(&s_ticket2, 1);
                if (k >= ntops) break;
                int v = leafq[k], sp;
                if (v == 0) {
                    sp = t.span[0];
                    v = hv[0];
                } else {
                    const int u0 = t.par[v];
                    while (*(volatile uint8_t*)&sready[u0] == 0) __nanosleep(20);
                    __threadfence_block();
                    sp = *(volatile uint8_t*)&t.span[u0];
                }
                while (v != 0xFFFF) {
                    sp = smap[(size_t)v * MSB + sp];
                    t.span[v] = (uint8_t)sp;
                    if (cs[v + 1] - cs[v] > 1) {   // light children start paths below v
                        __threadfence_block();
                        *(volatile uint8_t*)&sready[v] = 1;
                    }
                    v = hv[v];
                }
            }
        }
        __syncthreads();
        FMARK(4);
        // ---- segment records, outputs and S6
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
                const uint32_t e = t.E[i * ES + l];
                if (l >= lo && l <= hi && e < be) { be = e; lt = l; }   // smallest l attaining the min (R11)
            }
            const int ls = t.recE[i * ES + lt];
            const bool straight = (t.x[i] == t.x[u]) || (t.y[i] == t.y[u]);
            const uint32_t s = seg_bend(wh->h.dir[ls], wh->h.dir[lt], straight) | ((uint32_t)ls << 8) |
                               ((uint32_t)lt << 16) | ((uint32_t)straight << 24);
            if (o.rec_seg) o.rec_seg[o.rec_off[o.list_base + blockIdx.x] + i] = s;
            else o.seg[a0 + i] = s;
            if (commit) commit_edge(g, &wh->h, t.x[i], t.y[i], t.x[u], t.y[u], s, hyb_z(hy, a0 + i, s, LT));
        }
    } else {
        if (lane == 0) {
            for (;;) {
                const int k = atomicAdd(&s_ticket2, 1);
                if (k >= ntops) break;
                int v = leafq[k], sp;
                if (v == 0) {
                    sp = t.span[0];
                    v = hv[0];
                } else {
                    const int u0 = t.par[v];
                    while (*(volatile uint8_t*)&sready[u0] == 0) __nanosleep(20);
                    __threadfence_block();
                    sp = *(volatile uint8_t*)&t.span[u0];
                }
                uint32_t e[ES];
                {
                    const uint4* ep = reinterpret_cast<const uint4*>(t.E + v * ES);
#pragma unroll
                    for (int q = 0; q < ES / 4; q++) {
                        const uint4 w = ep[q];
                        e[4 * q] = w.x; e[4 * q + 1] = w.y; e[4 * q + 2] = w.z; e[4 * q + 3] = w.w;
                    }
                }
                for (;;) {
                    const int u = t.par[v];
                    const int nx = hv[v];
                    const int nc = cs[v + 1] - cs[v];
                    uint32_t en[ES];   // prefetch the next node's E row while this node's argmins resolve
                    {
                        const uint4* ep = reinterpret_cast<const uint4*>(t.E + (nx == 0xFFFF ? v : nx) * ES);
#pragma unroll
                        for (int q = 0; q < ES / 4; q++) {
                            const uint4 w = ep[q];
                            en[4 * q] = w.x; en[4 * q + 1] = w.y; en[4 * q + 2] = w.z; en[4 * q + 3] = w.w;
                        }
                    }
                    const int lo = sp >> 4, hi = sp & 15;
                    uint32_t be = 0xFFFFFFFFu;
                    int lt = lo;
#pragma unroll
                    for (int l = 0; l < LT; l++)
                        if (l >= lo && l <= hi && e[l] < be) { be = e[l]; lt = l; }   // smallest l attaining the min (R11)
                    const int ls = t.recE[v * ES + lt];
                    sp = t.recB[v * ES + ls];
                    const bool straight = (t.x[v] == t.x[u]) || (t.y[v] == t.y[u]);
                    const uint32_t bend = seg_bend(wh->h.dir[ls], wh->h.dir[lt], straight);
                    t.seg[v] = bend | ((uint32_t)ls << 8) | ((uint32_t)lt << 16) | ((uint32_t)straight << 24);
                    if (nc > 1) {   // light children start paths below v: publish its span
                        t.span[v] = (uint8_t)sp;
                        __threadfence_block();
                        *(volatile uint8_t*)&sready[v] = 1;
                    }
                    if (nx == 0xFFFF) break;
                    v = nx;
#pragma unroll
                    for (int q = 0; q < ES; q++) e[q] = en[q];
                }
            }
        }
        __syncthreads();
        FMARK(4);
        // ---- outputs and S6
        for (int i = 1 + tid; i < m; i += T) {
            const uint32_t s = t.seg[i];
            if (o.rec_seg) o.rec_seg[o.rec_off[o.list_base + blockIdx.x] + i] = s;
            else o.seg[a0 + i] = s;
            if (commit) {
                const int u = t.par[i];
                commit_edge(g, &wh->h, t.x[i], t.y[i], t.x[u], t.y[u], s, hyb_z(hy, a0 + i, s, LT));
            }
        }
    }
    if (tid == 0) {
        if (o.rec_seg) { o.rec_seg[o.rec_off[o.list_base + blockIdx.x]] = 0xFFFFFFFFu; o.rec_cost[o.list_base + blockIdx.x] = s_cost; }
        else { o.seg[a0] = 0xFFFFFFFFu; o.cost[net] = s_cost; }
    }
#ifdef FGR_TIMING
    FMARK(5);
    if (tid == 0 && m > 600)
        printf("FLOW m=%d K=%d fast=%lld inline=%lld wstate=%lld wlight=%lld prologue=%lld gather=%lld forward=%lld backtrack=%lld commit=%lld\n", m, K,
               s_wst[0], s_wst[1], s_wst[2], s_wst[3], tm[1] - tm[0], tm[2] - tm[1], tm[3] - tm[2], tm[4] - tm[3], tm[5] - tm[4]);
#endif
#undef FMARK
}

template <int LT, int WARPS>
cudaError_t launch_flow(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                        const Out& o, bool commit, const Prep& prep) {
    const size_t smem = a16(sizeof(WHdr)) + flow_bytes(maxm, LT, WARPS);
    static bool configured = false;
    if (!configured) {
        cudaFuncAttributes fa;
        cudaError_t e = cudaFuncGetAttributes(&fa, k_dp_flow<LT, WARPS>);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(k_dp_flow<LT, WARPS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     g->max_smem - (int)fa.sharedSizeBytes);
        if (e != cudaSuccess) return e;
        configured = true;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(n);
    cfg.blockDim = dim3(32 * WARPS);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k_dp_flow<LT, WARPS>, g->view, nv, list, n, o, commit ? 1 : 0, prep, g->hy.view());
}

constexpr int kWalkWarpsS = 4;   // warps per CTA, nets of 3..8 nodes
constexpr int kWalkWarpsL = 2;   // warps per CTA, nets of 9..32 nodes

template <int LT, int MC, int WARPS>
cudaError_t launch_walk(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, const Out& o,
                        bool commit) {
    const size_t smem = a16(sizeof(WHdr)) + (size_t)WARPS * WK<LT>::G * wtabs_bytes(MC, LT);
    static bool configured = false;
    if (!configured) {
        cudaError_t e = cudaFuncSetAttribute(k_dp_walk<LT, MC, WARPS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)smem);
        if (e != cudaSuccess) return e;
        configured = true;
    }
    const int per_cta = WARPS * WK<LT>::G;
    k_dp_walk<LT, MC, WARPS><<<(n + per_cta - 1) / per_cta, 32 * WARPS, smem, st>>>(g->view, nv, list, n, o, commit ? 1 : 0,
                                                                                 g->hy.view());
    return cudaGetLastError();
}

}  // namespace

// Nets of 3..mc nodes (mc = FGR_MID_NET or FGR_SMALL_NET) through the walk kernel.
cudaError_t fgr_launch_walk(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int mc,
                            const Out& o, bool commit) {
    if (n <= 0) return cudaSuccess;
    switch (g->L) {
#define FGR_LT(L)                                                                                              \
    case L:                                                                                                    \
        return mc <= FGR_MID_NET ? launch_walk<L, FGR_MID_NET, kWalkWarpsS>(g, st, nv, list, n, o, commit)   \
                                 : launch_walk<L, FGR_SMALL_NET, kWalkWarpsL>(g, st, nv, list, n, o, commit);
        FGR_LT(2) FGR_LT(3) FGR_LT(4) FGR_LT(5) FGR_LT(6) FGR_LT(7) FGR_LT(8) FGR_LT(9) FGR_LT(10) FGR_LT(11)
        FGR_LT(12) FGR_LT(13) FGR_LT(14) FGR_LT(15) FGR_LT(16)
#undef FGR_LT
        default: return cudaErrorInvalidValue;
    }
}

// Largest net the flow kernel holds (8 warps), and the launcher (4 warps up to 128 nodes).
int fgr_flow_max_nodes(const fgr_grid* g) {
    int m = 4096;
    while (m > FGR_SMALL_NET && a16(sizeof(WHdr)) + flow_bytes(m, g->L, 8) + 256 > (size_t)g->max_smem) m -= 8;
    return m;
}

cudaError_t fgr_launch_flow(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                            const Out& o, bool commit, const Prep& prep) {
    if (n <= 0) return cudaSuccess;
    switch (g->L) {
#define FGR_LT(L)                                                                                                   \
    case L:                                                                                                         \
        return maxm <= 128 ? launch_flow<L, 4>(g, st, nv, list, n, maxm, o, commit, prep)                          \
                           : launch_flow<L, 8>(g, st, nv, list, n, maxm, o, commit, prep);
        FGR_LT(2) FGR_LT(3) FGR_LT(4) FGR_LT(5) FGR_LT(6) FGR_LT(7) FGR_LT(8) FGR_LT(9) FGR_LT(10) FGR_LT(11)
        FGR_LT(12) FGR_LT(13) FGR_LT(14) FGR_LT(15) FGR_LT(16)
#undef FGR_LT
        default: return cudaErrorInvalidValue;
    }
}
