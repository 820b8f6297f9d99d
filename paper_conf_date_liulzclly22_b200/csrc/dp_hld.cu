// dp_hld.cu — S4 tree DP + S5 backtrack + S6 commit for nets of more than
// FGR_SMALL_NET nodes, organised along a heavy-path decomposition of the tree
// (SURVEY.md §8(a)).
//
// The recurrences are those of dp.cu (§III-D, Eqs. (1)-(7), L582-756;
// the generalised Eq. (4) at the root, reading R9).  For a non-root node v with
// heavy child h (largest subtree), light children Λ and pin span [plo, phi]:
//     K_v(lo,hi) = V(lo,hi) + Σ_{c∈Λ} min_{l∈[lo,hi]} E_c(l)
//     G_v(a,b)   = min_{lo<=a, hi>=b} K_v(lo,hi)                    (dominance minimum)
//     B_v(ls)    = min_l [E_h(l) + G_v(A(min(ls,l)), B(max(ls,l)))]  (Eq. (2) by span enumeration, R3)
//     E_v(lt)    = min_ls [C_v(ls,lt) + B_v(ls)]                    (Eqs. (1),(3): both bends, R5)
// with A(x) = min(x, plo), B(x) = max(x, phi) (identity without pins).  For a
// node without light children G_v = V, so
//     B_v(ls) = min( min_{l<=ls}[E_h(l) - V0(A(l))] + V0(B(ls)),  min_{l>=ls}[E_h(l) + V0(B(l))] - V0(A(ls)) )
// (V0(x) = viapre[x]): a prefix and a suffix minimum, O(L) instead of O(L^2).  The
// same split, on packed (value, lo, hi) keys, gives the R11 argmin spans.
//
// The paper evaluates a net's nodes in DFS order with one block per net and the
// L "parallel computation flows" in its threads (P:L320-333, L698-705,
// L754-756): the critical path is the tree depth times one node step.  Here:
//   P1  the leg costs of every edge are gathered at once (costs are fixed in a batch);
//   P2  leaves get their E vector, one thread per leaf;
//   P3  heavy paths are walked bottom-up, one lane group (lane = layer) per path,
//       all paths of one light depth at once (<= log2(m) + 1 rounds); a branching
//       node's G_v is built first (its light children are final);
//   P4  one thread per node recomputes B_v with R11 argmin keys from the final
//       E vectors, the E_v argmins, and folds them into a byte table
//       phi_v[parent span] = span of v;
//   P5  the top-down backtrack (S5) is one byte load per node along each path;
//   P6  outputs and the S6 commit, one thread per edge.
// One CTA per net (a persistent grid loops over the launch's nets).  Per-node
// tables live in shared memory when they fit (nets up to ~1100 nodes at L = 9),
// otherwise in a per-CTA global workspace; G tables of branching nodes always live
// in the global workspace (L2).  Nets of up to 65535 nodes are accepted.
#include <cub/cub.cuh>

#include "dp_common.cuh"

#ifdef FGR_HLD_TIMING
#define HMARK(i) do { if (threadIdx.x == 0) tmk[i] = clock64(); } while (0)
#else
#define HMARK(i) do { } while (0)
#endif

namespace {

constexpr int kHldMaxRounds = 17;     // light depth <= log2(65535) + 1

__host__ __device__ constexpr int hld_ns(int LT) { return LT * (LT + 1) / 2; }

// triangular span index: row lo holds hi = lo..LT-1
__host__ __device__ __forceinline__ int tri_idx(int LT, int lo, int hi) { return lo * LT - (lo * (lo - 1)) / 2 + (hi - lo); }

// edge type byte: 0 bent L, 1 straight H (y_v == y_u), 2 straight V, 3 hybrid (L + Z transfer matrix)
enum { ET_BENT = 0, ET_SH = 1, ET_SV = 2, ET_HYB = 3 };

struct HldTabs {
    // small (shared memory unless the net is huge)
    uint16_t* par;     // 0xFFFF at the root
    uint16_t* hv;      // heavy child, 0xFFFF = leaf
    uint16_t* pn;      // path nodes (bottom -> head), paths deepest light depth first
    uint16_t* po;      // [npaths + 1]
    uint16_t* cs;      // [m + 1] child CSR
    uint16_t* cl;      // [m]
    uint16_t* bl;      // [m] branching nodes (>= 2 children) grouped by round (light depth of their path)
    int8_t* plo;
    int8_t* phi;
    uint8_t* et;       // edge type of the node's edge to its parent
    uint8_t* span;     // chosen via span of the node (triangular index)
    uint8_t* recE;     // [m][LT] argmin ls of E_v(lt)
    uint8_t* phit;     // [m][NS] span of v (tri index) for each span of its parent (tri index)
    // bulk (shared memory when it fits)
    uint32_t* E;       // [m][LT]
    uint32_t* LG;      // [m][2][LT] leg 1 by ls (H on row y_v / V on col x_v), leg 2 by lt (V on col x_u / H on row y_u)
    // global workspace
    unsigned long long* GK;   // [m][NS] packed G_v keys of branching nodes (and a branching root)
    uint32_t* MX;             // [m][LT(l)][LT(lt)] transfer matrices M_v(lt, l) of non-leaf nodes
};

__host__ __device__ inline size_t hld_small_bytes(int m, int LT) {
    return 4 * a16((size_t)(m + 1) * 2) + 3 * a16((size_t)m * 2) + 4 * a16((size_t)m) + a16((size_t)m * LT) +
           a16((size_t)m * hld_ns(LT));
}
__host__ __device__ inline size_t hld_bulk_bytes(int m, int LT) {
    return a16((size_t)m * LT * 4) + a16((size_t)m * 2 * LT * 4);
}
__host__ __device__ inline size_t hld_gk_bytes(int m, int LT) {
    return a16((size_t)m * hld_ns(LT) * 8) + a16((size_t)m * LT * LT * 4);   // GK + MX
}

__device__ inline void hld_carve_small(HldTabs& t, unsigned char* p, int m, int LT) {
    t.par = (uint16_t*)p; p += a16((size_t)(m + 1) * 2);
    t.hv = (uint16_t*)p; p += a16((size_t)(m + 1) * 2);
    t.po = (uint16_t*)p; p += a16((size_t)(m + 1) * 2);
    t.cs = (uint16_t*)p; p += a16((size_t)(m + 1) * 2);
    t.pn = (uint16_t*)p; p += a16((size_t)m * 2);
    t.cl = (uint16_t*)p; p += a16((size_t)m * 2);
    t.bl = (uint16_t*)p; p += a16((size_t)m * 2);
    t.plo = (int8_t*)p; p += a16((size_t)m);
    t.phi = (int8_t*)p; p += a16((size_t)m);
    t.et = p; p += a16((size_t)m);
    t.span = p; p += a16((size_t)m);
    t.recE = p; p += a16((size_t)m * LT);
    t.phit = p;
}
__device__ inline void hld_carve_bulk(HldTabs& t, unsigned char* p, int m, int LT) {
    t.E = (uint32_t*)p; p += a16((size_t)m * LT * 4);
    t.LG = (uint32_t*)p;
}

// Per-thread constants: viapre, zero-cost-run starts, direction mask.
template <int LT>
struct HldConst {
    uint32_t vp[LT];       // viapre[l]
    uint32_t zl[LT];       // zlo[l]: smallest lo with V(lo, l) == 0
    uint32_t hmask;        // layers with dir == H
    __device__ __forceinline__ void load(const Hdr* h) {
#pragma unroll
        for (int i = 0; i < LT; i++) { vp[i] = h->viapre[i]; zl[i] = h->zlo[i]; }
        hmask = 0;
#pragma unroll
        for (int i = 0; i < LT; i++) hmask |= (h->dir[i] == 0 ? 1u : 0u) << i;
    }
    __device__ __forceinline__ bool is_h(int l) const { return (hmask >> l) & 1u; }
    __device__ __forceinline__ uint32_t V(int a, int b) const {   // a, b compile-time after unrolling
        return vp[a] >= vp[b] ? vp[a] - vp[b] : vp[b] - vp[a];
    }
};

// Gather of one leg: cost of positions a..b on `line` of direction d for every layer of
// that direction, written to dst[layer] (exact uint32 differences of the segmented prefix, R19).
__device__ __forceinline__ void hld_gather(const DirView& d, int line, int a, int b, uint32_t* dst, const uint8_t* los) {
    const size_t pa = ((size_t)line * d.len + a) * d.W, pb = ((size_t)line * d.len + b) * d.W;
    const size_t sa = ((size_t)line * d.nseg + (a >> FGR_SEG_SHIFT)) * d.W;
    const size_t sb = ((size_t)line * d.nseg + (b >> FGR_SEG_SHIFT)) * d.W;
    const int nq = d.W >> 2;
#pragma unroll
    for (int q = 0; q < 4; q++) {
        if (q < nq) {
            const uint4 Pa = __ldg(reinterpret_cast<const uint4*>(d.P + pa) + q);
            const uint4 Pb = __ldg(reinterpret_cast<const uint4*>(d.P + pb) + q);
            const uint4 Sa = __ldg(reinterpret_cast<const uint4*>(d.SB + sa) + q);
            const uint4 Sb = __ldg(reinterpret_cast<const uint4*>(d.SB + sb) + q);
            if (4 * q + 0 < d.cnt) dst[los[4 * q + 0]] = (Sb.x + Pb.x) - (Sa.x + Pa.x);
            if (4 * q + 1 < d.cnt) dst[los[4 * q + 1]] = (Sb.y + Pb.y) - (Sa.y + Pa.y);
            if (4 * q + 2 < d.cnt) dst[los[4 * q + 2]] = (Sb.z + Pb.z) - (Sa.z + Pa.z);
            if (4 * q + 3 < d.cnt) dst[los[4 * q + 3]] = (Sb.w + Pb.w) - (Sa.w + Pa.w);
        }
    }
}

// C_v(ls, lt) (FGR_INF = no route) for compile-time ls, lt:
//   straight edge (reading R7): one leg on ls = lt of the edge's direction;
//   bent L edge (R5): leg 1 on ls, bend via V(ls, lt), leg 2 on lt, directions differing;
//   hybrid edge (NEXT #1): the precomputed L+Z transfer matrix M_e[lt][ls].
template <int LT>
__device__ __forceinline__ uint32_t hld_cost(const HldConst<LT>& c, int et, const uint32_t* l1, const uint32_t* l2,
                                             const uint32_t* hm, int ls, int lt) {
    if (et == ET_HYB) return hm[lt * LT + ls];
    if (et == ET_BENT) return c.is_h(ls) != c.is_h(lt) ? sat_add(sat_add(l1[ls], c.V(ls, lt)), l2[lt]) : FGR_INF;
    const bool hdir = et == ET_SH;
    return (ls == lt && c.is_h(lt) == hdir) ? l1[lt] : FGR_INF;
}

// C_v(ls, lt) for every ls and a runtime lt (one thread's row): see hld_cost.
template <int LT>
__device__ __forceinline__ void hld_cost_row(const HldConst<LT>& c, int et, const uint32_t* lg, const uint32_t* hm, int lt,
                                             uint32_t (&cc)[LT]) {
    if (et == ET_HYB) {
#pragma unroll
        for (int ls = 0; ls < LT; ls++) cc[ls] = hm[lt * LT + ls];
        return;
    }
    uint32_t vt = 0;
#pragma unroll
    for (int i = 0; i < LT; i++) vt = (i == lt) ? c.vp[i] : vt;
    const bool th = c.is_h(lt);
    if (et == ET_BENT) {
        const uint32_t l2 = lg[LT + lt];
#pragma unroll
        for (int ls = 0; ls < LT; ls++) {
            const uint32_t vv = c.vp[ls] >= vt ? c.vp[ls] - vt : vt - c.vp[ls];
            cc[ls] = c.is_h(ls) != th ? sat_add(sat_add(lg[ls], vv), l2) : FGR_INF;
        }
        return;
    }
    const uint32_t leg = (th == (et == ET_SH)) ? lg[lt] : FGR_INF;
#pragma unroll
    for (int ls = 0; ls < LT; ls++) cc[ls] = (ls == lt) ? leg : FGR_INF;
}

// Packed dominance table of node v from its light children, built by one warp (lane = lo,
// then lane = b) in its scratch R and copied to GK[v]: key(a,b) = min over lo <= a, hi >= b of
// (K_v(lo,hi) << 8 | lo << 4 | hi), stored at the triangular index of (a, b).
template <int LT>
__device__ __forceinline__ void hld_build_G(const HldConst<LT>& c, const HldTabs& t, unsigned long long* R, int v,
                                            int lane) {
    const bool on = lane < LT;
    const int lo = on ? lane : 0;
    if (on) {
        const int hvv = t.hv[v];
        const int k0 = t.cs[v], k1 = t.cs[v + 1];
        uint32_t acc[LT];
        uint32_t vpl = 0;
#pragma unroll
        for (int i = 0; i < LT; i++) vpl = (i == lo) ? c.vp[i] : vpl;
#pragma unroll
        for (int hi = 0; hi < LT; hi++) acc[hi] = hi >= lo ? c.vp[hi] - vpl : FGR_INF;
        for (int k = k0; k < k1; k++) {
            const int ch = t.cl[k];
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
                R[lo * LT + hi] = run;
            }
    }
    __syncwarp();
    if (on) {
        const int bcol = lane;
        unsigned long long pr = ~0ull;
        unsigned long long* gk = t.GK + (size_t)v * hld_ns(LT);
#pragma unroll
        for (int a = 0; a < LT; a++)
            if (a <= bcol) {
                const unsigned long long x = R[a * LT + bcol];
                pr = x < pr ? x : pr;
                R[a * LT + bcol] = pr;
                gk[tri_idx(LT, a, bcol)] = pr;
            }
    }
    __syncwarp();
}

// ---------------------------------------------------------------- the kernel
template <int LT, bool SM>
__global__ void __launch_bounds__(512, 1) k_dp_hld(GridView g, NetsView nv, const int32_t* __restrict__ list, int count,
                                                   Out o, int commit, HldPrep hp, HybView hy, unsigned char* gws,
                                                   size_t gws_stride, int mode) {
    constexpr int GPW = groups_of(LT);
    constexpr int NS = hld_ns(LT);
    extern __shared__ __align__(16) unsigned char smem[];
    Hdr* h = reinterpret_cast<Hdr*>(smem);
    __shared__ uint8_t s_los[2][FGR_MAXL];
    __shared__ uint8_t s_tlo[NS], s_thi[NS];
    __shared__ int s_rb[kHldMaxRounds + 1];
    __shared__ int s_bro[kHldMaxRounds + 2], s_bcur[kHldMaxRounds + 1];
    __shared__ unsigned long long s_root;
    const int tid = threadIdx.x, T = blockDim.x;
    const int warp = tid >> 5, lane = lane_id();
    const int gi = lane / LT;
    const bool glane = gi < GPW;
    const int gl = glane ? lane - gi * LT : 0;
    const int gbase = glane ? gi * LT : 0;
    unsigned char* sp = smem + a16(sizeof(Hdr));
    unsigned long long* R = reinterpret_cast<unsigned long long*>(sp) + (size_t)warp * LT * LT;   // per warp
    sp += a16((size_t)(T >> 5) * LT * LT * 8);
    init_hdr(h, g);
    for (int i = tid; i < 2 * FGR_MAXL; i += T) s_los[i / FGR_MAXL][i % FGR_MAXL] = g.layer_of_slot[i / FGR_MAXL][i % FGR_MAXL];
    for (int lo = 0; lo < LT; lo++)
        for (int hi = lo + tid; hi < LT; hi += T) { s_tlo[tri_idx(LT, lo, hi)] = (uint8_t)lo; s_thi[tri_idx(LT, lo, hi)] = (uint8_t)hi; }
    __syncthreads();
    unsigned char* gslot = gws + (size_t)blockIdx.x * gws_stride;
    bool waited = false;

    for (int idx = blockIdx.x; idx < count; idx += gridDim.x) {
#ifdef FGR_HLD_TIMING
        long long tmk[12];
        long long t3a = 0, t3b = 0, tx = 0, trb[8] = {0, 0, 0, 0, 0, 0, 0, 0}, tra[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        int rlen[8] = {0, 0, 0, 0, 0, 0, 0, 0};
#endif
        HMARK(0);
        const int net = list[idx];
        const int a0 = nv.off[net];
        const int m = nv.off[net + 1] - a0;
        const int info = hp.info[net];
        const int np = info & 0xFFFF, nr = info >> 16;
        const int hnet = hy.net ? hy.net[net] : -1;
        HldTabs t;
        {
            unsigned char* gp = gslot;
            t.GK = reinterpret_cast<unsigned long long*>(gp);
            t.MX = reinterpret_cast<uint32_t*>(gp + a16((size_t)m * NS * 8));
            gp += hld_gk_bytes(m, LT);
            if (SM) {   // every per-net table in shared memory (mode 0): plain LDS/STS addressing
                hld_carve_small(t, sp, m, LT);
                hld_carve_bulk(t, sp + a16(hld_small_bytes(m, LT)), m, LT);
            } else if (mode == 2) {
                hld_carve_small(t, gp, m, LT);
                hld_carve_bulk(t, gp + a16(hld_small_bytes(m, LT)), m, LT);
            } else {
                hld_carve_small(t, sp, m, LT);
                hld_carve_bulk(t, mode == 0 ? sp + a16(hld_small_bytes(m, LT)) : gp, m, LT);
            }
        }
        // ---- P0: tree and decomposition (demand-independent)
        for (int i = tid; i < m; i += T) {
            int et = ET_BENT;
            if (i) {
                const int u = nv.par[a0 + i];
                t.par[i] = (uint16_t)u;
                const int xv = nv.x[a0 + i], yv = nv.y[a0 + i], xu = nv.x[a0 + u], yu = nv.y[a0 + u];
                et = (yv == yu) ? ET_SH : (xv == xu) ? ET_SV : ET_BENT;
                if (et == ET_BENT && hnet >= 0 && hy.slot[a0 + i] >= 0) et = ET_HYB;
            } else {
                t.par[0] = 0xFFFF;
            }
            t.et[i] = (uint8_t)et;
            t.plo[i] = nv.plo[a0 + i];
            t.phi[i] = nv.phi[a0 + i];
            t.hv[i] = hp.hv[a0 + i];
            t.pn[i] = hp.pn[a0 + i];
            t.cs[i] = hp.cs[a0 + i];
            if (i + 1 < m) t.cl[i] = hp.cl[a0 + i];
        }
        for (int q = tid; q < np; q += T) {
            t.po[q] = hp.po[a0 + q];
            const int r = hp.pr[a0 + q];
            if (q == 0 || hp.pr[a0 + q - 1] != r) s_rb[r] = q;
        }
        if (tid == 0) { t.po[np] = (uint16_t)m; t.cs[m] = (uint16_t)(m - 1); }
        if (tid <= kHldMaxRounds) s_bcur[tid] = 0;
        __syncthreads();
        // branching nodes (the root included) by round = light depth: count, offsets, scatter
        for (int v = tid; v < m; v += T)
            if (t.cs[v + 1] - t.cs[v] >= 2) atomicAdd(&s_bcur[hp.ld[a0 + v]], 1);
        __syncthreads();
        if (tid == 0) {
            int acc = 0;
            for (int r = 0; r < nr; r++) { s_bro[r] = acc; acc += s_bcur[r]; s_bcur[r] = s_bro[r]; }
            s_bro[nr] = acc;
        }
        __syncthreads();
        for (int v = tid; v < m; v += T)
            if (t.cs[v + 1] - t.cs[v] >= 2) t.bl[atomicAdd(&s_bcur[hp.ld[a0 + v]], 1)] = (uint16_t)v;
        if (!waited) { pdl_wait(); waited = true; }   // the refresh must be done before the gathers
        __syncthreads();
        HMARK(1);
        // ---- P1: leg gathers (costs are fixed during the batch): 4 tasks per edge
        //   0: leg 1 H on row y_v, 1: leg 1 V on col x_v, 2: leg 2 V on col x_u, 3: leg 2 H on row y_u
        for (int task = tid; task < 4 * (m - 1); task += T) {
            const int v = 1 + (task >> 2), type = task & 3;
            const int et = t.et[v];
            if (et == ET_HYB || (et == ET_SH && type != 0) || (et == ET_SV && type != 1)) continue;
            const int u = t.par[v];
            const int xv = nv.x[a0 + v], yv = nv.y[a0 + v], xu = nv.x[a0 + u], yu = nv.y[a0 + u];
            uint32_t* dst = t.LG + (size_t)v * 2 * LT + (type >= 2 ? LT : 0);
            if (type == 0) hld_gather(g.h, yv, min(xv, xu), max(xv, xu), dst, s_los[0]);
            else if (type == 1) hld_gather(g.v, xv, min(yv, yu), max(yv, yu), dst, s_los[1]);
            else if (type == 2) hld_gather(g.v, xu, min(yv, yu), max(yv, yu), dst, s_los[1]);
            else hld_gather(g.h, yu, min(xv, xu), max(xv, xu), dst, s_los[0]);
        }
        __syncthreads();
        HMARK(2);
        // ---- P2: leaves get E_v, single-child nodes their matrix M_v; one lane group per node
        // (lane = lt), the warp's groups in lockstep:
        //   leaf:   E_v(lt)   = min_ls C_v(ls,lt) + V(A(ls), B(ls))
        //   chain:  M_v(lt,l) = min( V0(B(l)) + min_{ls<=l}[C(ls,lt) - V0(A(ls))],  min_{ls>=l}[C(ls,lt) + V0(B(ls))] - V0(A(l)) )
        {
            HldConst<LT> c;
            c.load(h);
            const uint32_t VPM = c.vp[LT - 1];
            for (int base = 1 + warp * GPW; base < m; base += (T >> 5) * GPW) {
                const int v = base + gi;
                if (!glane || v >= m) continue;
                const int nch = t.cs[v + 1] - t.cs[v];
                if (nch >= 2) continue;
                const int lt = gl;
                const int et = t.et[v];
                const int plo = t.plo[v], phi = t.phi[v];
                const bool pin = plo >= 0;
                uint32_t cc[LT];
                hld_cost_row<LT>(c, et, t.LG + (size_t)v * 2 * LT,
                                 et == ET_HYB ? hy.M + (size_t)hy.slot[a0 + v] * LT * LT : nullptr, lt, cc);
                const uint32_t vpl = pin ? h->viapre[plo] : 0u, vph = pin ? h->viapre[phi] : 0u;
                uint32_t vA[LT], vB[LT];
#pragma unroll
                for (int l = 0; l < LT; l++) {
                    vA[l] = (pin && l > plo) ? vpl : c.vp[l];
                    vB[l] = (pin && l < phi) ? vph : c.vp[l];
                }
                if (nch == 0) {
                    uint32_t best = FGR_INF;
#pragma unroll
                    for (int ls = 0; ls < LT; ls++) best = min(best, sat_add(cc[ls], vB[ls] - vA[ls]));
                    t.E[(size_t)v * LT + lt] = best;
                } else {
                    uint32_t P[LT];
                    uint32_t run = 0xFFFFFFFFu;
#pragma unroll
                    for (int l = 0; l < LT; l++) {   // C(ls,lt) + VPM - vA[ls], prefix min over ls <= l (INF stays >= INF)
                        run = min(run, cc[l] + (VPM - vA[l]));
                        P[l] = run;
                    }
                    run = 0xFFFFFFFFu;
                    uint32_t* mx = t.MX + (size_t)v * LT * LT + lt;
#pragma unroll
                    for (int l = LT - 1; l >= 0; l--) {   // C(ls,lt) + vB[ls], suffix min over ls >= l
                        run = min(run, cc[l] + vB[l]);
                        mx[l * LT] = min(min(P[l] + vB[l] - VPM, run - vA[l]), FGR_INF);
                    }
                }
            }
        }
        __syncthreads();
        HMARK(3);
        // ---- P3: light-depth rounds, deepest first
        for (int r = nr - 1; r >= 0; r--) {
#ifdef FGR_HLD_TIMING
            if (threadIdx.x == 0) tx = clock64();
#endif
            const int q0 = s_rb[r], q1 = r > 0 ? s_rb[r - 1] : np;
            const int k0 = t.po[q0], k1 = t.po[q1];
            // P3a: G tables and transfer matrices of this round's branching nodes (their light
            // children are final), one warp per node: lanes = lo / b for G, then the 81 entries of M
            {
                HldConst<LT> c;
                c.load(h);
                for (int bi = s_bro[r] + warp; bi < s_bro[r + 1]; bi += (T >> 5)) {
                    const int v = t.bl[bi];
                    hld_build_G<LT>(c, t, R, v, lane);
                    if (v == 0) continue;   // the root has no edge (its G serves the final Eq. (4) step)
                    const int et = t.et[v];
                    const int plo = t.plo[v], phi = t.phi[v];
                    const bool pin = plo >= 0;
                    const uint32_t* lg = t.LG + (size_t)v * 2 * LT;
                    const uint32_t* hm = et == ET_HYB ? hy.M + (size_t)hy.slot[a0 + v] * LT * LT : nullptr;
                    uint32_t* mx = t.MX + (size_t)v * LT * LT;
                    for (int en = lane; en < LT * LT; en += 32) {   // M_v(lt,l) = min_ls C(ls,lt) + G_v(A(min(ls,l)), B(max(ls,l)))
                        const int l = en / LT, lt = en - l * LT;
                        uint32_t cc[LT];
                        hld_cost_row<LT>(c, et, lg, hm, lt, cc);
                        uint32_t best = FGR_INF;
#pragma unroll
                        for (int ls = 0; ls < LT; ls++) {
                            int a = min(ls, l), b = max(ls, l);
                            if (pin) { a = min(a, plo); b = max(b, phi); }
                            best = min(best, sat_add(cc[ls], (uint32_t)(R[a * LT + b] >> 8)));
                        }
                        mx[en] = best;
                    }
                    __syncwarp();   // R is reused by the warp's next node
                }
            }
            __syncthreads();
#ifdef FGR_HLD_TIMING
            if (threadIdx.x == 0) { t3a += clock64() - tx; if (r < 8) tra[r] = clock64() - tx; tx = clock64(); }
#endif
            // P3b: walk this round's paths bottom-up.  A warp walks GPW paths in lockstep (one lane
            // group per path, lane = layer; full-warp shuffles, no divergence between the groups):
            // E_v(lt) = min_l M_v(lt,l) + E_h(l), the rows of the next four matrices in flight.
            for (int base = q0 + warp * GPW; base < q1; base += (T >> 5) * GPW) {
                const int q = base + gi;
                const bool act = glane && q < q1;
                int kb = 0, nsteps = 0;
                uint32_t e = 0;
                if (act) {
                    kb = t.po[q];
                    const int ke = t.po[q + 1];
                    const int kend = t.pn[ke - 1] == 0 ? ke - 1 : ke;   // the root has no edge
                    nsteps = kend - kb - 1;
                    e = t.E[(size_t)t.pn[kb] * LT + gl];                // the bottom is a leaf (P2)
                }
                const int maxs = __reduce_max_sync(0xffffffffu, (unsigned)nsteps);
                uint32_t m0[LT], m1[LT], m2[LT], m3[LT], m4[LT], m5[LT], m6[LT], m7[LT];
                auto ldm = [&](int i, uint32_t(&mr)[LT]) {
                    if (i < nsteps) {
                        const uint32_t* mx = t.MX + (size_t)t.pn[kb + 1 + i] * LT * LT + gl;
#pragma unroll
                        for (int l = 0; l < LT; l++) mr[l] = mx[l * LT];
                    }
                };
                auto step = [&](int i, const uint32_t(&mr)[LT]) {
                    uint32_t ev[LT];
#pragma unroll
                    for (int l = 0; l < LT; l++) ev[l] = sat_add(__shfl_sync(0xffffffffu, e, gbase + l), mr[l]);
#pragma unroll
                    for (int s2 = 1; s2 < LT; s2 <<= 1)
#pragma unroll
                        for (int i2 = 0; i2 + s2 < LT; i2 += 2 * s2) ev[i2] = min(ev[i2], ev[i2 + s2]);
                    if (i < nsteps) {
                        e = ev[0];
                        t.E[(size_t)t.pn[kb + 1 + i] * LT + gl] = e;
                    }
                };
                ldm(0, m0); ldm(1, m1); ldm(2, m2); ldm(3, m3); ldm(4, m4); ldm(5, m5); ldm(6, m6); ldm(7, m7);
                for (int i = 0; i < maxs; i += 8) {
                    step(i, m0); ldm(i + 8, m0);
                    if (i + 1 >= maxs) break;
                    step(i + 1, m1); ldm(i + 9, m1);
                    if (i + 2 >= maxs) break;
                    step(i + 2, m2); ldm(i + 10, m2);
                    if (i + 3 >= maxs) break;
                    step(i + 3, m3); ldm(i + 11, m3);
                    if (i + 4 >= maxs) break;
                    step(i + 4, m4); ldm(i + 12, m4);
                    if (i + 5 >= maxs) break;
                    step(i + 5, m5); ldm(i + 13, m5);
                    if (i + 6 >= maxs) break;
                    step(i + 6, m6); ldm(i + 14, m6);
                    if (i + 7 >= maxs) break;
                    step(i + 7, m7); ldm(i + 15, m7);
                }
            }
            __syncthreads();
#ifdef FGR_HLD_TIMING
            if (threadIdx.x == 0) {
                t3b += clock64() - tx;
                if (r < 8) {
                    trb[r] = clock64() - tx;
                    int mx = 0;
                    for (int q = q0; q < q1; q++) mx = max(mx, t.po[q + 1] - t.po[q]);
                    rlen[r] = mx;
                }
            }
#endif
        }
        HMARK(4);
        // ---- P4: argmins (R11 order) and the backtrack tables; one lane group per node, the warp's
        // groups in lockstep (full-warp shuffles): lane = ls for the B_v keys, lane = lt for the E_v
        // argmins, lane = lo for the phi rows
        if (tid == 0) {
            // generalised Eq. (4) at the root: min over l of E_h(l) + G(hull({l} + pins)) (any span for a Steiner root)
            const int nch = t.cs[1] - t.cs[0];
            const int plo = t.plo[0], phi = t.phi[0];
            const int ra = plo >= 0 ? plo : LT - 1, rb = plo >= 0 ? phi : 0;
            const uint32_t* Eh = t.E + (size_t)t.hv[0] * LT;
            const unsigned long long* gk = t.GK;
            unsigned long long best = ~0ull;
            for (int l = 0; l < LT; l++) {
                const int a = min(ra, l), b = max(rb, l);
                const unsigned long long gkey = nch >= 2 ? gk[tri_idx(LT, a, b)]
                    : ((unsigned long long)(h->viapre[b] - h->viapre[a]) << 8) | (unsigned)(h->zlo[a] << 4) | (unsigned)b;
                const unsigned long long key = ((unsigned long long)sat_add(Eh[l], (uint32_t)(gkey >> 8)) << 8) | (gkey & 0xFFull);
                best = key < best ? key : best;
            }
            s_root = best;
        }
        {
            HldConst<LT> c;
            c.load(h);
            const uint32_t VPM = c.vp[LT - 1];
            for (int base = 1 + warp * GPW; base < m; base += (T >> 5) * GPW) {
                const int vq = base + gi;
                const bool act = glane && vq < m;
                const int v = act ? vq : 1;
                const int nch = t.cs[v + 1] - t.cs[v];
                const int plo = t.plo[v], phi = t.phi[v];
                const bool pin = plo >= 0;
                const int ls = gl;
                // B_v(ls) key: (value, lo, hi) minimal (R11)
                unsigned long long kb;
                const uint32_t vpl = pin ? h->viapre[plo] : 0u, vph = pin ? h->viapre[phi] : 0u;
                const uint32_t zpl = pin ? h->zlo[plo] : 0u;
                uint32_t vA[LT], vB[LT], zA[LT], bI[LT];   // V0(A(l)), V0(B(l)), zlo(A(l)), B(l)
#pragma unroll
                for (int l = 0; l < LT; l++) {
                    const bool ca = pin && l > plo, cb = pin && l < phi;
                    vA[l] = ca ? vpl : c.vp[l];
                    vB[l] = cb ? vph : c.vp[l];
                    zA[l] = ca ? zpl : c.zl[l];
                    bI[l] = cb ? (uint32_t)phi : (uint32_t)l;
                }
                uint32_t vAs = 0, vBs = 0, zAs = 0, bIs = 0;   // the same at l = ls
#pragma unroll
                for (int l = 0; l < LT; l++)
                    if (l == ls) { vAs = vA[l]; vBs = vB[l]; zAs = zA[l]; bIs = bI[l]; }
                if (nch == 0) {
                    kb = ((unsigned long long)(vBs - vAs) << 8) | (zAs << 4) | bIs;
                } else if (nch == 1) {
                    // l >= ls: value E_h(l) + V0(B(l)) - V0(A(ls)), span (zlo(A(ls)), B(l))
                    // l <= ls: value E_h(l) - V0(A(l)) + V0(B(ls)), span (zlo(A(l)), B(ls))
                    const uint32_t* Eh = t.E + (size_t)t.hv[v] * LT;
                    unsigned long long k1 = ~0ull, k2 = ~0ull;
#pragma unroll
                    for (int l = 0; l < LT; l++) {
                        const uint32_t e = Eh[l];
                        const unsigned long long a1 = ((unsigned long long)(e + vB[l]) << 8) | bI[l];
                        const unsigned long long a2 = ((unsigned long long)(e + (VPM - vA[l])) << 8) | (zA[l] << 4);
                        if (l >= ls) k1 = a1 < k1 ? a1 : k1;
                        if (l <= ls) k2 = a2 < k2 ? a2 : k2;
                    }
                    const unsigned long long x1 = (k1 - ((unsigned long long)vAs << 8)) | (zAs << 4);
                    const unsigned long long x2 = (k2 + ((unsigned long long)vBs << 8) - ((unsigned long long)VPM << 8)) | bIs;
                    kb = x1 < x2 ? x1 : x2;
                } else {
                    const uint32_t* Eh = t.E + (size_t)t.hv[v] * LT;
                    const unsigned long long* gk = t.GK + (size_t)v * NS;
                    int a0s = ls, b0s = ls;
                    if (pin) { a0s = min(a0s, plo); b0s = max(b0s, phi); }
                    kb = ~0ull;
#pragma unroll
                    for (int l = 0; l < LT; l++) {
                        const unsigned long long gkey = gk[tri_idx(LT, min(a0s, l), max(b0s, l))];
                        const unsigned long long key = ((unsigned long long)sat_add(Eh[l], (uint32_t)(gkey >> 8)) << 8) | (gkey & 0xFFull);
                        kb = key < kb ? key : kb;
                    }
                }
                const uint32_t bv = (uint32_t)min(kb >> 8, (unsigned long long)FGR_INF);
                const int cd = (int)(kb & 0xFF);
                const int mycode = tri_idx(LT, cd >> 4, cd & 15);
                // E_v argmin for lt = gl: smallest ls minimising B(ls) + C(ls, lt)
                const int et = t.et[v];
                uint32_t cc[LT];
                hld_cost_row<LT>(c, et, t.LG + (size_t)v * 2 * LT,
                                 et == ET_HYB ? hy.M + (size_t)hy.slot[a0 + v] * LT * LT : nullptr, gl, cc);
                uint32_t best = FGR_INF;
                int bls = gl;
#pragma unroll
                for (int l = 0; l < LT; l++) {
                    const uint32_t cst = sat_add(__shfl_sync(0xffffffffu, bv, gbase + l), cc[l]);
                    if (cst < best) { best = cst; bls = l; }
                }
                const int sol = __shfl_sync(0xffffffffu, mycode, gbase + bls);
                // phi row lo = gl: child layer = smallest l in [lo, hi] minimising E_v(l) (R11)
                const uint32_t* Ev = t.E + (size_t)v * LT;
                uint8_t* ph = t.phit + (size_t)v * NS;
                uint32_t be = FGR_INF;
                int cur = 0;
#pragma unroll
                for (int hi = 0; hi < LT; hi++) {
                    const int sh = __shfl_sync(0xffffffffu, sol, gbase + hi);
                    const uint32_t ev = Ev[hi];
                    if (hi == gl || (hi > gl && ev < be)) { be = ev; cur = sh; }
                    if (act && hi >= gl) ph[tri_idx(LT, gl, hi)] = (uint8_t)cur;
                }
                if (act) t.recE[(size_t)v * LT + gl] = (uint8_t)bls;
            }
        }
        __syncthreads();
        HMARK(5);
        // ---- P5: top-down backtrack (S5), one thread per path, shallowest light depth first
        if (tid == 0) {
            const int cd = (int)(s_root & 0xFF);
            t.span[0] = (uint8_t)tri_idx(LT, cd >> 4, cd & 15);
        }
        __syncthreads();
        for (int r = 0; r < nr; r++) {
            const int q0 = s_rb[r], q1 = r > 0 ? s_rb[r - 1] : np;
            for (int q = q0 + tid; q < q1; q += T) {
                const int kb = t.po[q], ke = t.po[q + 1];
                int k = ke - 1;
                int v = t.pn[k];
                int s;
                if (v == 0) s = t.span[0];
                else { s = t.phit[(size_t)v * NS + t.span[t.par[v]]]; t.span[v] = (uint8_t)s; }
                for (k = ke - 2; k >= kb; k--) {
                    v = t.pn[k];
                    s = t.phit[(size_t)v * NS + s];
                    t.span[v] = (uint8_t)s;
                }
            }
            __syncthreads();
        }
        HMARK(6);
        // ---- P6: outputs and the S6 commit, one thread per edge
        for (int i = 1 + tid; i < m; i += T) {
            const int u = t.par[i];
            const int su = t.span[u];
            const int lo = s_tlo[su], hi = s_thi[su];
            const uint32_t* Ei = t.E + (size_t)i * LT;
            uint32_t be = Ei[lo];
            int lt = lo;
            for (int l = lo + 1; l <= hi; l++) {
                const uint32_t e = Ei[l];
                if (e < be) { be = e; lt = l; }
            }
            const int ls = t.recE[(size_t)i * LT + lt];
            const int et = t.et[i];
            const bool straight = et == ET_SH || et == ET_SV;
            const uint32_t bend = seg_bend(h->dir[ls], h->dir[lt], straight);
            const uint32_t s = bend | ((uint32_t)ls << 8) | ((uint32_t)lt << 16) | ((uint32_t)straight << 24);
            if (o.rec_seg) o.rec_seg[o.rec_off[o.list_base + idx] + i] = s;
            else o.seg[a0 + i] = s;
            if (commit)
                commit_edge(g, h, nv.x[a0 + i], nv.y[a0 + i], nv.x[a0 + u], nv.y[a0 + u], s, hyb_z(hy, a0 + i, s, LT));
        }
        if (tid == 0) {
            const uint32_t total = (uint32_t)(s_root >> 8);
            if (o.rec_seg) { o.rec_seg[o.rec_off[o.list_base + idx]] = 0xFFFFFFFFu; o.rec_cost[o.list_base + idx] = total; }
            else { o.seg[a0] = 0xFFFFFFFFu; o.cost[net] = total; }
        }
        __syncthreads();
        HMARK(7);
#ifdef FGR_HLD_TIMING
        if (threadIdx.x == 0 && m > 500)
            printf("HLD m=%d np=%d nr=%d mode=%d load=%lld gather=%lld p2=%lld p3a=%lld p3b=%lld p4=%lld p5=%lld p6=%lld total=%lld\n",
                   m, np, nr, mode, tmk[1] - tmk[0], tmk[2] - tmk[1], tmk[3] - tmk[2], t3a, t3b, tmk[5] - tmk[4],
                   tmk[6] - tmk[5], tmk[7] - tmk[6], tmk[7] - tmk[0]);
        if (threadIdx.x == 0 && m > 900)
            printf("HLDR m=%d r0 len=%d a=%lld b=%lld | r1 len=%d a=%lld b=%lld | r2 len=%d a=%lld b=%lld | r3 len=%d a=%lld b=%lld | r4 len=%d a=%lld b=%lld\n",
                   m, rlen[0], tra[0], trb[0], rlen[1], tra[1], trb[1], rlen[2], tra[2], trb[2], rlen[3], tra[3], trb[3],
                   rlen[4], tra[4], trb[4]);
#endif
    }
}

// ---------------------------------------------------------------- decomposition (once per stage)
// One CTA per net.  Scratch per node (shared memory, or a global slot for huge nets):
// sub (subtree size), hk (heavy key), cnt (child count / cursor), ld (light depth),
// hd / len (path head and length by path position).
constexpr int kPrepT = 256;

__host__ __device__ inline size_t hprep_bytes(int m) { return 8 * a16((size_t)(m + 1) * 4) + a16((size_t)m + 1); }
constexpr int kLeafOrderMax = 4096;   // nets up to this size get the deepest-first leaf order (k_dp_tree)

__global__ void __launch_bounds__(kPrepT) k_hld_prep(NetsView nv, const int32_t* __restrict__ list, uint16_t* hv_o,
                                                     uint16_t* cs_o, uint16_t* cl_o, uint16_t* pn_o, uint16_t* po_o,
                                                     uint8_t* pr_o, int32_t* info_o, uint8_t* ld_o, uint16_t* lf_o,
                                                     unsigned char* gtmp,
                                                     size_t gstride, int smem_cap) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ int s_cnt[kHldMaxRounds + 1], s_start[kHldMaxRounds + 1], s_nr, s_np;
    using Scan = cub::BlockScan<int, kPrepT>;
    __shared__ typename Scan::TempStorage s_scan;
    __shared__ int s_carry;
    const int net = list[blockIdx.x];
    const int a0 = nv.off[net], m = nv.off[net + 1] - a0;
    const int tid = threadIdx.x;
    unsigned char* base = (int)hprep_bytes(m) <= smem_cap ? smem : gtmp + (size_t)blockIdx.x * gstride;
    int* sub = (int*)base;
    unsigned* hk = (unsigned*)(base + a16((size_t)(m + 1) * 4));
    int* cnt = (int*)(base + 2 * a16((size_t)(m + 1) * 4));
    int* hd = (int*)(base + 3 * a16((size_t)(m + 1) * 4));
    int* len = (int*)(base + 4 * a16((size_t)(m + 1) * 4));
    int* par = (int*)(base + 5 * a16((size_t)(m + 1) * 4));
    int* dep = (int*)(base + 6 * a16((size_t)(m + 1) * 4));
    unsigned* lk = (unsigned*)(base + 7 * a16((size_t)(m + 1) * 4));
    uint8_t* ld = base + 8 * a16((size_t)(m + 1) * 4);
    for (int i = tid; i < m; i += kPrepT) { sub[i] = 1; hk[i] = 0; cnt[i] = 0; par[i] = nv.par[a0 + i]; }
    if (tid <= kHldMaxRounds) s_cnt[tid] = 0;
    __syncthreads();
    if (tid == 0) {
        for (int i = m - 1; i >= 1; i--) sub[par[i]] += sub[i];
    }
    for (int i = 1 + tid; i < m; i += kPrepT) atomicAdd(&cnt[par[i]], 1);
    __syncthreads();
    // heavy child: largest subtree, ties to the smallest index
    for (int i = 1 + tid; i < m; i += kPrepT) atomicMax(&hk[par[i]], ((unsigned)sub[i] << 16) | (0xFFFFu - (unsigned)i));
    // child CSR starts: exclusive scan of the child counts
    if (tid == 0) s_carry = 0;
    __syncthreads();
    for (int b0 = 0; b0 < m; b0 += kPrepT) {
        const int i = b0 + tid;
        const int x = i < m ? cnt[i] : 0;
        int ex, tot;
        Scan(s_scan).ExclusiveSum(x, ex, tot);
        if (i < m) { cs_o[a0 + i] = (uint16_t)(s_carry + ex); cnt[i] = s_carry + ex; }   // cnt becomes the fill cursor
        __syncthreads();
        if (tid == 0) s_carry += tot;
        __syncthreads();
    }
    for (int v = tid; v < m; v += kPrepT) hv_o[a0 + v] = hk[v] ? (uint16_t)(0xFFFFu - (hk[v] & 0xFFFFu)) : (uint16_t)0xFFFF;
    __syncthreads();
    for (int i = 1 + tid; i < m; i += kPrepT) cl_o[a0 + atomicAdd(&cnt[par[i]], 1)] = (uint16_t)i;
    if (tid == 0) {
        // light depth: a light edge adds one (parent index < child index: one forward pass)
        ld[0] = 0;
        dep[0] = 0;
        int mx = 0;
        for (int i = 1; i < m; i++) {
            const int p = par[i];
            dep[i] = dep[p] + 1;
            const int hvp = hk[p] ? (int)(0xFFFFu - (hk[p] & 0xFFFFu)) : -1;
            const int d = ld[p] + (hvp != i ? 1 : 0);
            ld[i] = (uint8_t)d;
            mx = d > mx ? d : mx;
        }
        s_nr = mx + 1;
    }
    __syncthreads();
    // path heads: the root and every light child; count per light depth
    for (int v = tid; v < m; v += kPrepT) {
        bool head = v == 0;
        if (!head) {
            const int p = par[v];
            head = (int)(0xFFFFu - (hk[p] & 0xFFFFu)) != v;
        }
        if (head) atomicAdd(&s_cnt[ld[v]], 1);
    }
    __syncthreads();
    if (tid == 0) {
        int acc = 0;
        for (int r = s_nr - 1; r >= 0; r--) { s_start[r] = acc; acc += s_cnt[r]; s_cnt[r] = 0; }
        s_np = acc;
    }
    __syncthreads();
    for (int v = tid; v < m; v += kPrepT) {
        bool head = v == 0;
        if (!head) {
            const int p = par[v];
            head = (int)(0xFFFFu - (hk[p] & 0xFFFFu)) != v;
        }
        if (!head) continue;
        int n = 1, w = v;
        while (hk[w]) { w = (int)(0xFFFFu - (hk[w] & 0xFFFFu)); n++; }
        const int q = s_start[ld[v]] + atomicAdd(&s_cnt[ld[v]], 1);
        hd[q] = v;
        len[q] = n;
    }
    __syncthreads();
    const int np = s_np;
    if (tid == 0) s_carry = 0;
    __syncthreads();
    for (int b0 = 0; b0 < np; b0 += kPrepT) {
        const int q = b0 + tid;
        const int x = q < np ? len[q] : 0;
        int ex, tot;
        Scan(s_scan).ExclusiveSum(x, ex, tot);
        if (q < np) { sub[q] = s_carry + ex; po_o[a0 + q] = (uint16_t)(s_carry + ex); pr_o[a0 + q] = ld[hd[q]]; }
        __syncthreads();
        if (tid == 0) s_carry += tot;
        __syncthreads();
    }
    for (int q = tid; q < np; q += kPrepT) {
        int w = hd[q];
        const int start = sub[q], n = len[q];
        for (int k = n - 1; k >= 0; k--) {
            pn_o[a0 + start + k] = (uint16_t)w;
            w = hk[w] ? (int)(0xFFFFu - (hk[w] & 0xFFFFu)) : -1;
        }
    }
    for (int v = tid; v < m; v += kPrepT) ld_o[a0 + v] = ld[v];
    if (tid == 0) info_o[net] = np | (s_nr << 16);
    // leaves (= path bottoms) deepest first, ties by index: the start order of k_dp_tree's
    // leaf-to-root dataflow (long chains start first)
    if (m > kLeafOrderMax) return;
    __syncthreads();
    for (int q = tid; q < np; q += kPrepT) {
        int w = hd[q];
        while (hk[w]) w = (int)(0xFFFFu - (hk[w] & 0xFFFFu));
        lk[q] = ((unsigned)(0xFFFF - dep[w]) << 16) | (unsigned)w;
    }
    __syncthreads();
    for (int q = tid; q < np; q += kPrepT) {
        const unsigned key = lk[q];
        int rank = 0;
        for (int j = 0; j < np; j++) rank += lk[j] < key;
        lf_o[a0 + rank] = (uint16_t)(key & 0xFFFFu);
    }
}

struct HldPlan {
    int T, mode, grid;
    size_t dyn, stride;
};

template <int LT>
HldPlan hld_plan(const fgr_grid* g, int n, int maxm) {
    HldPlan p;
    p.T = maxm > 128 ? 512 : 256;
    const size_t fixed = a16(sizeof(Hdr)) + a16((size_t)(p.T / 32) * LT * LT * 8);
    const size_t margin = 2048;   // static shared memory of the kernel
    const size_t sm = hld_small_bytes(maxm, LT);
    const size_t bk = hld_bulk_bytes(maxm, LT);
    const size_t cap = (size_t)g->max_smem;
    if (fixed + margin + sm + bk <= cap) { p.mode = 0; p.dyn = fixed + sm + bk; }
    else if (fixed + margin + sm <= cap) { p.mode = 1; p.dyn = fixed + sm; }
    else { p.mode = 2; p.dyn = fixed; }
    // persistent grid: at most two resident CTAs per SM (512-thread CTAs at <= 128 registers)
    p.grid = n < 2 * g->num_sms ? n : 2 * g->num_sms;
    p.stride = a16(hld_gk_bytes(maxm, LT) + (p.mode >= 1 ? a16(bk) : 0) + (p.mode == 2 ? a16(sm) : 0) + 256);
    return p;
}

template <int LT>
cudaError_t launch_hld_lt(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                          const Out& o, bool commit, const HldPrep& hp, unsigned char* ws) {
    static int configured = 0;
    if (!configured) {
        cudaFuncAttributes fa;
        cudaError_t e = cudaFuncGetAttributes(&fa, k_dp_hld<LT, true>);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(k_dp_hld<LT, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     g->max_smem - (int)fa.sharedSizeBytes - 64);
        if (e == cudaSuccess) e = cudaFuncGetAttributes(&fa, k_dp_hld<LT, false>);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(k_dp_hld<LT, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     g->max_smem - (int)fa.sharedSizeBytes - 64);
        if (e != cudaSuccess) return e;
        configured = 1;
    }
    const HldPlan p = hld_plan<LT>(g, n, maxm);
    if (!ws) return cudaErrorInvalidValue;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(p.grid);
    cfg.blockDim = dim3(p.T);
    cfg.dynamicSmemBytes = p.dyn;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    if (p.mode == 0)
        return cudaLaunchKernelEx(&cfg, k_dp_hld<LT, true>, g->view, nv, list, n, o, commit ? 1 : 0, hp, g->hy.view(), ws,
                                  p.stride, p.mode);
    return cudaLaunchKernelEx(&cfg, k_dp_hld<LT, false>, g->view, nv, list, n, o, commit ? 1 : 0, hp, g->hy.view(), ws,
                              p.stride, p.mode);
}

}  // namespace

size_t fgr_hld_ws_bytes(const fgr_grid* g, int n, int maxm) {
    if (n <= 0) return 0;
    HldPlan p{};
    switch (g->L) {
#define FGR_LT(k) case k: p = hld_plan<k>(g, n, maxm); break;
        FGR_LT(2) FGR_LT(3) FGR_LT(4) FGR_LT(5) FGR_LT(6) FGR_LT(7) FGR_LT(8) FGR_LT(9) FGR_LT(10) FGR_LT(11)
        FGR_LT(12) FGR_LT(13) FGR_LT(14) FGR_LT(15) FGR_LT(16)
#undef FGR_LT
        default: return 0;
    }
    return p.stride * (size_t)p.grid;
}

cudaError_t fgr_launch_hld(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                           const Out& o, bool commit, const HldPrep& hp, unsigned char* ws) {
    if (n <= 0) return cudaSuccess;
    switch (g->L) {
#define FGR_LT(k) case k: return launch_hld_lt<k>(g, st, nv, list, n, maxm, o, commit, hp, ws);
        FGR_LT(2) FGR_LT(3) FGR_LT(4) FGR_LT(5) FGR_LT(6) FGR_LT(7) FGR_LT(8) FGR_LT(9) FGR_LT(10) FGR_LT(11)
        FGR_LT(12) FGR_LT(13) FGR_LT(14) FGR_LT(15) FGR_LT(16)
#undef FGR_LT
        default: return cudaErrorInvalidValue;
    }
}

cudaError_t fgr_launch_hld_prep(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int count,
                                int maxm, uint16_t* hv, uint16_t* cs, uint16_t* cl, uint16_t* pn, uint16_t* po,
                                uint8_t* pr, int32_t* info, uint8_t* ld, uint16_t* lf) {
    if (count <= 0) return cudaSuccess;
    static int configured = 0;
    if (!configured) {
        cudaError_t e = cudaFuncSetAttribute(k_hld_prep, cudaFuncAttributeMaxDynamicSharedMemorySize, 160 * 1024);
        if (e != cudaSuccess) return e;
        configured = 1;
    }
    const int cap = 160 * 1024;
    const size_t need = hprep_bytes(maxm);
    unsigned char* gtmp = nullptr;
    size_t stride = 0;
    size_t dyn = need;
    if ((int)need > cap) {
        stride = a16(need);
        cudaError_t e;
        gtmp = (unsigned char*)fgr_scratch(g->s_hldt, stride * (size_t)count, &e);
        if (e != cudaSuccess) return e;
        dyn = cap;   // smaller nets of the launch still use shared memory
    }
    k_hld_prep<<<count, kPrepT, dyn, st>>>(nv, list, hv, cs, cl, pn, po, pr, info, ld, lf, gtmp, stride, (int)dyn);
    g->stats.kernel_launches++;
    return cudaGetLastError();
}
