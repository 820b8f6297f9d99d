// dp_tree.cu — S4 tree DP + S5 backtrack for nets of FGR_SMALL_NET+1 .. tree_cap(L)
// nodes (the large nets whose tables fit one SM's shared memory; bigger nets take
// k_dp_hld).  One CTA per net; the S6 commit of these nets runs afterwards in the
// grid-wide k_commit_nets so that a lone large net does not push its tens of
// thousands of unit-edge REDs through a single SM.
//
// Recurrences (§III-D, Eqs. (1)-(7), L582-756; readings R3, R5-R11 in
// DESIGN.md §3).  For node v with children Ch(v), pin span [plo, phi]:
//     F_v(lo,hi) = V(lo,hi) + Σ_{c∈Ch(v)} min_{l∈[lo,hi]} E_c(l)                  (Eq. (2), R3)
//     B_v(ls)    = min_{lo <= a(ls), hi >= b(ls)} F_v(lo,hi),  a = min(ls,plo), b = max(ls,phi)
//     E_v(lt)    = min_ls C_v(ls,lt) + B_v(ls)                                 (Eqs. (1),(3), R5, R7)
// and at the root the generalised Eq. (4) (R9): min over spans containing the pin span.
// With at most one child c the span minimum has the closed form
//     B_v(ls) = min_l E_c(l) + V(min(a,l), max(b,l))
//             = min_l E_c(l) + max(vp[b], vp[l]) - min(vp[a], vp[l])   (vp = via prefix, non-decreasing)
// (a leaf is the case E_c ≡ 0), and for a bent L edge (R5: ls and lt of different directions)
//     E_v(lt) = leg2(lt) + min_{ls: dir(ls) != dir(lt)} [B_v(ls) + leg1(ls) + |vp[ls] - vp[lt]|].
//
// Organisation (the paper's kernel walks a net's nodes in DFS order with one block per
// net and the L parallel computation flows in its threads):
//   P0  topology and the per-stage decomposition (k_hld_prep) into shared memory;
//   P1  every edge's leg costs gathered at once (costs are fixed during a batch);
//   P2  values, leaf-to-root dataflow: a lane group (lane = layer) takes leaves by ticket
//       (deepest first) and walks upwards; at a node with several children only the last
//       child to finish (pending-child counter) continues with the parent, so no group
//       ever waits and the critical path is the tree height, not a sum over levels;
//   P3  argmin tables in parallel over all nodes (R11 order): for every node the child
//       span phi_v[span of the parent] (the whole S5 decision for that edge) and recE;
//   P4  top-down backtrack along heavy paths (one byte load per node);
//   P5  outputs (seg, cost).
// All per-net tables live in shared memory at compile-time offsets (no pointer
// arithmetic in the hot loops), values are 32-bit with DPX min-plus (VIADDMNMX).
#include "dp_common.cuh"

#ifdef FGR_TREE_TIMING
__device__ __forceinline__ long long tclock() {   // clock read that stays between the barriers around it
    long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)::"memory");
    return t;
}
#define TMARK(i) do { if (threadIdx.x == 0) tmk[i] = tclock(); } while (0)
#else
#define TMARK(i) do { } while (0)
#endif

namespace {

constexpr int kTreeMaxRounds = 17;

__host__ __device__ constexpr int tr_ns(int LT) { return LT * (LT + 1) / 2; }
__host__ __device__ __forceinline__ int tr_tri(int LT, int lo, int hi) { return lo * LT - (lo * (lo - 1)) / 2 + (hi - lo); }
__host__ __device__ constexpr int tr_a16(int b) { return (b + 15) & ~15; }

enum { TE_BENT = 0, TE_SH = 1, TE_SV = 2, TE_HYB = 3 };

// Light-weight CTA-scope ordering (fence.sc, which __threadfence_block emits, is not needed here):
// the pending-child hand-off is one acq_rel atomic; publishing to the P3 queue is a release fence
// before the slot stores and an acquire fence after the consumer sees them.
__device__ __forceinline__ unsigned atom_dec_acqrel(unsigned* p) {
    unsigned old;
    asm volatile("atom.acq_rel.cta.shared::cta.add.u32 %0, [%1], %2;"
                 : "=r"(old)
                 : "r"((unsigned)__cvta_generic_to_shared(p)), "r"(0xFFFFFFFFu)
                 : "memory");
    return old;
}
__device__ __forceinline__ void fence_acqrel_cta() { asm volatile("fence.acq_rel.cta;" ::: "memory"); }

// CTA barrier after warp-divergent code: reconverge the warp first.  bar.sync counts a warp as
// arrived when its first lanes arrive, so without the __syncwarp a warp whose groups are still
// walking would let the CTA through (measured: P3 started while P2 was still running).
__device__ __forceinline__ void cta_sync() {
    __syncwarp();
    __syncthreads();
}

// Bytes of the shared-memory layout below (TL<LT, NT, CAP>::BYTES).
__host__ __device__ constexpr int tl_bytes(int LT, int NT, int CAP) {
    return 16 * CAP + 3 * tr_a16(4 * LT * CAP) + tr_a16(4 * CAP) + 4 * tr_a16(2 * CAP) + 2 * tr_a16(2 * CAP + 2) + tr_a16(tr_ns(LT) * CAP) +
           tr_a16(LT * CAP) + 4 * tr_a16(CAP) + tr_a16(2 * CAP) + (NT / 32) * groups_of(LT) * tr_a16(5 * LT * LT);
}

// Shared-memory layout for capacity CAP nodes (all offsets compile-time constants).
template <int LT, int NT, int CAP>
struct TL {
    static constexpr int NS = tr_ns(LT);
    static constexpr int GPW = groups_of(LT);
    static constexpr int NW = NT / 32;
    static constexpr int META = 0;                                // uint4 [CAP]  k0 | nch << 16, par | et << 16, vp[plo] (~0), vp[phi] (0)
    static constexpr int E = META + 16 * CAP;                     // uint32 [CAP][LT]  E_v(lt)
    static constexpr int LG1 = E + tr_a16(4 * LT * CAP);          // uint32 [CAP][LT]  leg 1 by ls (straight: the leg, INF off-direction)
    static constexpr int LG2 = LG1 + tr_a16(4 * LT * CAP);        // uint32 [CAP][LT]  leg 2 by lt
    static constexpr int PEND = LG2 + tr_a16(4 * LT * CAP);       // uint32 [CAP]      children still pending (P2)
    static constexpr int PAR = PEND + tr_a16(4 * CAP);            // uint16 [CAP]
    static constexpr int CS = PAR + tr_a16(2 * CAP);              // uint16 [CAP + 1]  child CSR
    static constexpr int CL = CS + tr_a16(2 * CAP + 2);           // uint16 [CAP]
    static constexpr int LF = CL + tr_a16(2 * CAP);               // uint16 [CAP]      leaves, deepest first
    static constexpr int PN = LF + tr_a16(2 * CAP);               // uint16 [CAP]      heavy-path nodes (bottom -> head)
    static constexpr int PO = PN + tr_a16(2 * CAP);               // uint16 [CAP + 1]  path starts
    static constexpr int PHI = PO + tr_a16(2 * CAP + 2);          // uint8 [CAP][NS]   span of v for each span of its parent
    static constexpr int RECE = PHI + tr_a16(NS * CAP);           // uint8 [CAP][LT]   argmin ls of E_v(lt)
    static constexpr int ET = RECE + tr_a16(LT * CAP);            // uint8 [CAP]       edge type
    static constexpr int PLO = ET + tr_a16(CAP);                  // int8 [CAP]
    static constexpr int PHIP = PLO + tr_a16(CAP);                // int8 [CAP]
    static constexpr int SPAN = PHIP + tr_a16(CAP);               // uint8 [CAP]       chosen span (S5)
    static constexpr int Q = SPAN + tr_a16(CAP);                  // uint16 [CAP]      finished nodes awaiting P3 (0xFFFF = empty)
    static constexpr int SCR = Q + tr_a16(2 * CAP);               // per group: uint32 [LT][LT] suffix minima + uint8 [LT][LT] argmin hi
    static constexpr int SCR_G = tr_a16(5 * LT * LT);
    static constexpr int BYTES = SCR + NW * GPW * SCR_G;
    static_assert(BYTES == tl_bytes(LT, NT, CAP), "layout size");
};

// Largest capacity of the 512-thread variant that fits the opt-in shared memory of an SM
// (227 KB less the kernel's static shared memory and a margin).
__host__ __device__ constexpr int tree_cap_nt(int LT, int NT) {
    int cap = 4096;
    while (cap > 64 && tl_bytes(LT, NT, cap) + 4096 > 227 * 1024) cap -= 16;
    return cap;
}
constexpr int kTreeBigNT = 384;   // threads of the variant for the largest nets (up to 168 registers per thread)
__host__ __device__ constexpr int tree_cap512(int LT) { return tree_cap_nt(LT, kTreeBigNT); }

template <int LT>
struct Lane {                       // per-lane constants of a lane group (lane = layer gl)
    int gl, gbase;
    unsigned gmask;
    uint32_t myvp;                  // vp[gl]
    uint32_t D[LT];                 // |vp[ls] - vp[gl]| if dir(ls) != dir(gl), else INF  (bent-edge via + direction rule)
};

template <int LT>
__device__ __forceinline__ Lane<LT> make_lane(const GridView& g, uint32_t hmask, int gl, int gbase, unsigned gmask) {
    Lane<LT> ln;
    ln.gl = gl;
    ln.gbase = gbase;
    ln.gmask = gmask;
    ln.myvp = 0;
#pragma unroll
    for (int l = 0; l < LT; l++) ln.myvp = (l == gl) ? g.viapre[l] : ln.myvp;
    const bool myh = (hmask >> gl) & 1u;
#pragma unroll
    for (int l = 0; l < LT; l++) {
        const uint32_t vl = g.viapre[l];
        const bool lh = (hmask >> l) & 1u;
        ln.D[l] = lh != myh ? (vl >= ln.myvp ? vl - ln.myvp : ln.myvp - vl) : FGR_INF;
    }
    return ln;
}

// C_v argmin / values for a hybrid edge: M[lt][ls] (transfer matrix of the L + Z candidates).
template <int LT>
__device__ __forceinline__ const uint32_t* hyb_row(const HybView& hy, int gnode, int lt) {
    return hy.M + ((size_t)hy.slot[gnode] * LT + lt) * LT;
}


// Shared-memory views of one net's tables (compile-time offsets).
template <int LT, int NT, int CAP>
struct TV {
    using T = TL<LT, NT, CAP>;
    unsigned char* sm;
    __device__ __forceinline__ uint32_t* E() const { return reinterpret_cast<uint32_t*>(sm + T::E); }
    __device__ __forceinline__ uint32_t* LG1() const { return reinterpret_cast<uint32_t*>(sm + T::LG1); }
    __device__ __forceinline__ uint32_t* LG2() const { return reinterpret_cast<uint32_t*>(sm + T::LG2); }
    __device__ __forceinline__ uint16_t* CS() const { return reinterpret_cast<uint16_t*>(sm + T::CS); }
    __device__ __forceinline__ uint16_t* CL() const { return reinterpret_cast<uint16_t*>(sm + T::CL); }
    __device__ __forceinline__ uint8_t* PHI() const { return sm + T::PHI; }
    __device__ __forceinline__ uint8_t* RECE() const { return sm + T::RECE; }
    __device__ __forceinline__ uint8_t* ET() const { return sm + T::ET; }
    __device__ __forceinline__ int8_t* PLO() const { return reinterpret_cast<int8_t*>(sm + T::PLO); }
    __device__ __forceinline__ int8_t* PHIP() const { return reinterpret_cast<int8_t*>(sm + T::PHIP); }
};

// P2, span-table part of a node step for a node with several children (or the root): lane lo
// builds F(lo, hi) over all children (the child prev from X, the others from shared memory), then
// B(ls) = min_{lo <= a} min_{hi >= b} F(lo, hi).  At the root it stores the generalised Eq. (4)
// minimum and its span in root_out[1], root_out[0] instead (R9, R11).
template <int LT, int NT, int CAP>
__device__ __forceinline__ uint32_t tree_multi_B(const GridView& g, unsigned char* sm, const Lane<LT>& ln, int v, int prev,
                                                 const uint32_t (&X)[LT], uint32_t* scrF, uint32_t* root_out) {
    const TV<LT, NT, CAP> t{sm};
    const uint32_t* sE = t.E();
    const int k0 = t.CS()[v], k1 = t.CS()[v + 1];
    const int plo = t.PLO()[v], phi = t.PHIP()[v];
    const bool pin = plo >= 0;
    uint32_t acc[LT];
#pragma unroll
    for (int hi = 0; hi < LT; hi++) acc[hi] = hi >= ln.gl ? g.viapre[hi] - ln.myvp : FGR_INF;
    for (int k = k0; k < k1; k++) {
        const int c = t.CL()[k];
        uint32_t run = FGR_INF;
        if (c == prev) {
#pragma unroll
            for (int hi = 0; hi < LT; hi++) {
                run = min(run, hi >= ln.gl ? X[hi] : FGR_INF);
                acc[hi] = sat_add(acc[hi], run);
            }
        } else {
            const uint32_t* Ec = sE + c * LT;
#pragma unroll
            for (int hi = 0; hi < LT; hi++) {
                run = min(run, hi >= ln.gl ? Ec[hi] : FGR_INF);
                acc[hi] = sat_add(acc[hi], run);
            }
        }
    }
    if (v == 0) {
        // first (lo, hi) in lexicographic order among the minimal spans containing the root's pin
        // span (any span for a Steiner root)
        const int ra = pin ? plo : LT - 1, rb = pin ? phi : 0;
        uint32_t bv = FGR_INF, bh = 0;
#pragma unroll
        for (int hi = LT - 1; hi >= 0; hi--)
            if (hi >= rb && acc[hi] <= bv) { bv = acc[hi]; bh = (uint32_t)hi; }
        if (ln.gl > ra) bv = FGR_INF;
        uint32_t best = FGR_INF, blo = 0, bhi = 0;
#pragma unroll
        for (int lo = 0; lo < LT; lo++) {
            const uint32_t x = __shfl_sync(ln.gmask, bv, ln.gbase + lo);
            const uint32_t h = __shfl_sync(ln.gmask, bh, ln.gbase + lo);
            if (x < best) { best = x; blo = (uint32_t)lo; bhi = h; }
        }
        if (ln.gl == 0) { root_out[0] = (uint32_t)tr_tri(LT, (int)blo, (int)bhi); root_out[1] = best; }
        return 0;
    }
    uint32_t run = FGR_INF;
#pragma unroll
    for (int b = LT - 1; b >= 0; b--) {
        run = min(run, acc[b]);
        scrF[ln.gl * LT + b] = run;
    }
    __syncwarp(ln.gmask);
    const int a = pin ? min(ln.gl, plo) : ln.gl, b = pin ? max(ln.gl, phi) : ln.gl;
    uint32_t B = FGR_INF;
#pragma unroll
    for (int lo = 0; lo < LT; lo++)
        if (lo <= a) B = min(B, scrF[lo * LT + b]);
    __syncwarp(ln.gmask);
    return B;
}

// P3 for node v (E of v and of its children final): recE_v and the phi table (R11 order).
template <int LT, int NT, int CAP>
__device__ __forceinline__ void tree_node_argmin(const GridView& g, const HybView& hy, unsigned char* sm,
                                                 const Lane<LT>& ln, int v, int a0, uint32_t* scrF) {
    constexpr int NS = tr_ns(LT);
    const TV<LT, NT, CAP> t{sm};
    const uint32_t* sE = t.E();
    uint8_t* scrH = reinterpret_cast<uint8_t*>(scrF + LT * LT);
    const int k0 = t.CS()[v], k1 = t.CS()[v + 1];
    const int plo = t.PLO()[v], phi = t.PHIP()[v];
    const bool pin = plo >= 0;
    // F row lo = gl, then suffix minima over hi with the smallest attaining hi
    uint32_t acc[LT];
#pragma unroll
    for (int hi = 0; hi < LT; hi++) acc[hi] = hi >= ln.gl ? g.viapre[hi] - ln.myvp : FGR_INF;
    for (int k = k0; k < k1; k++) {
        const uint32_t* Ec = sE + t.CL()[k] * LT;
        uint32_t run = FGR_INF;
#pragma unroll
        for (int hi = 0; hi < LT; hi++) {
            run = min(run, hi >= ln.gl ? Ec[hi] : FGR_INF);
            acc[hi] = sat_add(acc[hi], run);
        }
    }
    {
        uint32_t run = 0xFFFFFFFFu, rh = 0;
#pragma unroll
        for (int b = LT - 1; b >= 0; b--) {
            if (acc[b] <= run) { run = acc[b]; rh = (uint32_t)b; }
            scrF[ln.gl * LT + b] = run;
            scrH[ln.gl * LT + b] = (uint8_t)rh;
        }
    }
    __syncwarp(ln.gmask);
    // B(ls) and its span: smallest lo (then that lo's smallest hi) among the minimal spans
    const int a = pin ? min(ln.gl, plo) : ln.gl, b = pin ? max(ln.gl, phi) : ln.gl;
    uint32_t B = FGR_INF;
    int blo = -1;
#pragma unroll
    for (int lo = 0; lo < LT; lo++) {
        const uint32_t f = scrF[lo * LT + b];
        if (lo <= a && f < B) { B = f; blo = lo; }
    }
    const int spanB = blo >= 0 ? tr_tri(LT, blo, scrH[blo * LT + b]) : 0;
    __syncwarp(ln.gmask);
    // recE(lt): smallest ls minimising B(ls) + C(ls, lt)
    const int et = t.ET()[v];
    int bls = 0;
    if (et == TE_BENT) {
        const uint32_t bp = sat_add(B, t.LG1()[v * LT + ln.gl]);
        uint32_t best = FGR_INF;
#pragma unroll
        for (int ls = 0; ls < LT; ls++) {
            const uint32_t x = __viaddmin_u32(__shfl_sync(ln.gmask, bp, ln.gbase + ls), ln.D[ls], FGR_INF);
            if (x < best) { best = x; bls = ls; }
        }
    } else if (et == TE_HYB) {
        const uint32_t* M = hyb_row<LT>(hy, a0 + v, ln.gl);
        uint32_t best = FGR_INF;
#pragma unroll
        for (int ls = 0; ls < LT; ls++) {
            const uint32_t x = sat_add(__shfl_sync(ln.gmask, B, ln.gbase + ls), __ldg(M + ls));
            if (x < best) { best = x; bls = ls; }
        }
    } else {
        bls = ln.gl;   // R7: one candidate, ls = lt
    }
    t.RECE()[v * LT + ln.gl] = (uint8_t)bls;
    // phi row lo = gl: child layer = smallest l in [lo, hi] minimising E_v(l) (R11), then its span
    const int sol = __shfl_sync(ln.gmask, spanB, ln.gbase + bls);
    const uint32_t* Ev = sE + v * LT;
    uint8_t* ph = t.PHI() + v * NS;
    uint32_t be = FGR_INF;
    int curs = 0;
#pragma unroll
    for (int hi = 0; hi < LT; hi++) {
        const int sh = __shfl_sync(ln.gmask, sol, ln.gbase + hi);
        const uint32_t ev = Ev[hi];
        if (hi == ln.gl || (hi > ln.gl && ev < be)) { be = ev; curs = sh; }
        if (hi >= ln.gl) ph[tr_tri(LT, ln.gl, hi)] = (uint8_t)curs;
    }
}

template <int LT, int NT, int CAP>
__global__ void __launch_bounds__(NT, (NT >= 384 ? 1 : (NT >= 256 ? 2 : 4)))
k_dp_tree(GridView g, NetsView nv, const int32_t* __restrict__ list, int count, Out o, HldPrep hp, HybView hy,
          const uint32_t* __restrict__ legs, int legs_maxm) {
    using T = TL<LT, NT, CAP>;
    constexpr int NS = T::NS, GPW = T::GPW, NW = T::NW;
    extern __shared__ __align__(16) unsigned char sm[];
    __shared__ uint8_t s_los[2][FGR_MAXL];
    __shared__ uint8_t s_tlo[NS], s_thi[NS];
    __shared__ int s_rb[kTreeMaxRounds + 1];
    __shared__ int s_ticket, s_qtail, s_qhead;
    __shared__ uint32_t s_root[2];   // span, cost
#ifdef FGR_TREE_TIMING
    __shared__ long long s_wt[2][NT / 32];
    __shared__ int s_p3done, s_viol;
#endif
    uint32_t* const sE = reinterpret_cast<uint32_t*>(sm + T::E);
    uint32_t* const sLG1 = reinterpret_cast<uint32_t*>(sm + T::LG1);
    uint32_t* const sLG2 = reinterpret_cast<uint32_t*>(sm + T::LG2);
    uint32_t* const sPEND = reinterpret_cast<uint32_t*>(sm + T::PEND);
    uint16_t* const sPAR = reinterpret_cast<uint16_t*>(sm + T::PAR);
    uint16_t* const sCS = reinterpret_cast<uint16_t*>(sm + T::CS);
    uint16_t* const sCL = reinterpret_cast<uint16_t*>(sm + T::CL);
    uint16_t* const sLF = reinterpret_cast<uint16_t*>(sm + T::LF);
    uint16_t* const sPN = reinterpret_cast<uint16_t*>(sm + T::PN);
    uint16_t* const sPO = reinterpret_cast<uint16_t*>(sm + T::PO);
    uint8_t* const sPHI = sm + T::PHI;
    uint8_t* const sRECE = sm + T::RECE;
    uint8_t* const sET = sm + T::ET;
    int8_t* const sPLO = reinterpret_cast<int8_t*>(sm + T::PLO);
    int8_t* const sPHIP = reinterpret_cast<int8_t*>(sm + T::PHIP);
    uint8_t* const sSPAN = sm + T::SPAN;
    uint16_t* const sQ = reinterpret_cast<uint16_t*>(sm + T::Q);
    uint4* const sMETA = reinterpret_cast<uint4*>(sm + T::META);

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = lane_id();
    const int gi = lane / LT;
    const bool glane = gi < GPW;
    uint32_t hmask = 0;
#pragma unroll
    for (int l = 0; l < LT; l++) hmask |= (g.dir[l] == 0 ? 1u : 0u) << l;
    // P3 lane groups: GPW groups of LT lanes per warp.  P2: one group per warp whose LT lanes are
    // mirrored over the whole warp (lane % LT), so a walking warp never diverges between groups.
    const Lane<LT> ln = make_lane<LT>(g, hmask, glane ? lane - gi * LT : 0, glane ? gi * LT : 0,
                                      glane ? (((1u << LT) - 1u) << (gi * LT)) : (1u << lane));
    const Lane<LT> l2 = make_lane<LT>(g, hmask, lane % LT, 0, 0xffffffffu);
    uint32_t* const scrF = reinterpret_cast<uint32_t*>(sm + T::SCR + (warp * GPW + (glane ? gi : 0)) * T::SCR_G);
    for (int i = tid; i < 2 * FGR_MAXL; i += NT) s_los[i / FGR_MAXL][i % FGR_MAXL] = g.layer_of_slot[i / FGR_MAXL][i % FGR_MAXL];
    for (int lo = 0; lo < LT; lo++)
        for (int hi = lo + tid; hi < LT; hi += NT) { s_tlo[tr_tri(LT, lo, hi)] = (uint8_t)lo; s_thi[tr_tri(LT, lo, hi)] = (uint8_t)hi; }
    bool waited = false;

    for (int idx = blockIdx.x; idx < count; idx += gridDim.x) {
#ifdef FGR_TREE_TIMING
        long long tmk[8];
#endif
        TMARK(0);
        const int net = list[idx];
        const int a0 = nv.off[net];
        const int m = nv.off[net + 1] - a0;
        const int info = hp.info[net];
        const int np = info & 0xFFFF, nr = info >> 16;   // np = number of heavy paths = number of leaves
        const int hnet = hy.net ? hy.net[net] : -1;
        // ---- P0: topology (demand-independent: overlaps the refresh under PDL)
        for (int i = tid; i < m; i += NT) {
            int et = TE_BENT;
            int u = 0xFFFF;
            if (i) {
                u = nv.par[a0 + i];
                const int xv = nv.x[a0 + i], yv = nv.y[a0 + i], xu = nv.x[a0 + u], yu = nv.y[a0 + u];
                et = (yv == yu) ? TE_SH : (xv == xu) ? TE_SV : TE_BENT;
                if (et == TE_BENT && hnet >= 0 && hy.slot[a0 + i] >= 0) et = TE_HYB;
            }
            sPAR[i] = (uint16_t)u;
            sET[i] = (uint8_t)et;
            const int plo = nv.plo[a0 + i], phi = nv.phi[a0 + i];
            sPLO[i] = (int8_t)plo;
            sPHIP[i] = (int8_t)phi;
            const int c0 = hp.cs[a0 + i];
            const int c1 = i + 1 < m ? hp.cs[a0 + i + 1] : m - 1;
            sCS[i] = (uint16_t)c0;
            sMETA[i] = make_uint4((uint32_t)c0 | ((uint32_t)(c1 - c0) << 16), (uint32_t)u | ((uint32_t)et << 16),
                                  plo >= 0 ? g.viapre[plo] : 0xFFFFFFFFu, plo >= 0 ? g.viapre[phi] : 0u);
            sPEND[i] = (uint32_t)(c1 - c0);
            if (i + 1 < m) sCL[i] = hp.cl[a0 + i];
            sPN[i] = hp.pn[a0 + i];
            sQ[i] = 0xFFFF;
            if (i < np) { sLF[i] = hp.lf[a0 + i]; sPO[i] = hp.po[a0 + i]; }
            if (!legs && (et == TE_SH || et == TE_SV)) {   // the off-direction layers of a straight edge stay impossible (R6, R7)
#pragma unroll
                for (int l = 0; l < LT; l++) sLG1[i * LT + l] = FGR_INF;
            }
        }
        for (int q = tid; q < np; q += NT) {
            const int r = hp.pr[a0 + q];
            if (q == 0 || hp.pr[a0 + q - 1] != r) s_rb[r] = q;
        }
        if (tid == 0) { sCS[m] = (uint16_t)(m - 1); sPO[np] = (uint16_t)m; s_ticket = 0; s_qtail = 0; s_qhead = 0;
#ifdef FGR_TREE_TIMING
            s_p3done = 0; s_viol = 0;
#endif
        }
        if (!waited) { pdl_wait(); waited = true; }   // the refresh must be complete before the gathers
        cta_sync();
        TMARK(1);
        // ---- P1: leg costs.  Nets above 512 nodes: the rows k_tree_legs gathered with many SMs (LG1 |
        // LG2 blocks of legs_maxm rows); otherwise gathered here, 4 tasks per edge.
        if (legs) {
            const uint32_t* L1 = legs + (size_t)idx * 2 * legs_maxm * LT;
            const uint32_t* L2 = L1 + (size_t)legs_maxm * LT;
            for (int i = LT + tid; i < m * LT; i += NT) {
                sLG1[i] = __ldcg(L1 + i);
                sLG2[i] = __ldcg(L2 + i);
            }
        } else {
            // ---- P1: leg gathers, 4 tasks per edge:
            //   0: leg 1 H on row y_v, 1: leg 1 V on col x_v, 2: leg 2 V on col x_u, 3: leg 2 H on row y_u
#pragma unroll 4
            for (int task = tid; task < 4 * (m - 1); task += NT) {
                const int v = 1 + (task >> 2), type = task & 3;
                const int et = sET[v];
                if (et == TE_HYB || (et == TE_SH && type != 0) || (et == TE_SV && type != 1)) continue;
                const int u = sPAR[v];
                const int xv = nv.x[a0 + v], yv = nv.y[a0 + v], xu = nv.x[a0 + u], yu = nv.y[a0 + u];
                const bool H = type == 0 || type == 3;
                const int line = type == 0 ? yv : type == 1 ? xv : type == 2 ? xu : yu;
                const int pa = H ? min(xv, xu) : min(yv, yu);
                const int pb = H ? max(xv, xu) : max(yv, yu);
                const uint32_t* P = H ? g.h.P : g.v.P;
                const uint32_t* SB = H ? g.h.SB : g.v.SB;
                const int len = H ? g.h.len : g.v.len, W = H ? g.h.W : g.v.W, nseg = H ? g.h.nseg : g.v.nseg;
                const int cnt = H ? g.h.cnt : g.v.cnt;
                uint32_t* dst = (type >= 2 ? sLG2 : sLG1) + v * LT;
                const uint8_t* los = s_los[H ? 0 : 1];
                const size_t ia = ((size_t)line * len + pa) * W, ib = ((size_t)line * len + pb) * W;
                const size_t sa = ((size_t)line * nseg + (pa >> FGR_SEG_SHIFT)) * W;
                const size_t sb = ((size_t)line * nseg + (pb >> FGR_SEG_SHIFT)) * W;
                for (int q = 0; q < (W >> 2); q++) {
                    const uint4 Pa = __ldg(reinterpret_cast<const uint4*>(P + ia) + q);
                    const uint4 Pb = __ldg(reinterpret_cast<const uint4*>(P + ib) + q);
                    const uint4 Sa = __ldg(reinterpret_cast<const uint4*>(SB + sa) + q);
                    const uint4 Sb = __ldg(reinterpret_cast<const uint4*>(SB + sb) + q);
                    if (4 * q + 0 < cnt) dst[los[4 * q + 0]] = (Sb.x + Pb.x) - (Sa.x + Pa.x);
                    if (4 * q + 1 < cnt) dst[los[4 * q + 1]] = (Sb.y + Pb.y) - (Sa.y + Pa.y);
                    if (4 * q + 2 < cnt) dst[los[4 * q + 2]] = (Sb.z + Pb.z) - (Sa.z + Pa.z);
                    if (4 * q + 3 < cnt) dst[los[4 * q + 3]] = (Sb.w + Pb.w) - (Sa.w + Pa.w);
                }
            }
        }
        cta_sync();
        TMARK(2);
        // ---- P2 + P3: values (leaf-to-root dataflow, one walking group per warp) and, on warps
        // without forward work, the argmin tables of finished nodes (from the completion queue sQ).
        {
            int cur = -1;          // node of the warp's walk: -1 take a ticket, -2 no forward work left
            int prev = -1;         // node finished last (its E row is in X)
            uint32_t X[LT];        // E row of prev (every lane holds all of it)
            int nbuf = 0;          // finished nodes not yet published to sQ (lane % LT == i holds the i-th)
            int myid = 0;
            uint32_t* const scrW = reinterpret_cast<uint32_t*>(sm + T::SCR + warp * GPW * T::SCR_G);
#ifdef FGR_TREE_TIMING
            long long tst = 0, tmb = 0, tho = 0;
            int nst = 0, nmul = 0, nmb = 0;
#endif
            uint4 mv = make_uint4(0, 0, 0, 0);   // meta of cur
            uint32_t g1 = 0, g2 = 0;              // LG1 / LG2 of cur at layer gl
            while (true) {
                if (cur == -1) {
                    int t = 0;
                    if (lane == 0) t = atomicAdd(&s_ticket, 1);
                    t = __shfl_sync(0xffffffffu, t, 0);
                    if (t >= np) break;
                    cur = sLF[t];
                    mv = sMETA[cur];
                    g1 = sLG1[cur * LT + l2.gl];
                    g2 = sLG2[cur * LT + l2.gl];
                    prev = -1;
#ifdef FGR_TREE_TIMING
                    tst = clock64(); nst = 0; nmul = 0; tmb = 0; tho = 0; nmb = 0;
#endif
                }
                const int v = cur;
                const int u = (int)(mv.y & 0xFFFFu);
                const int nch = (int)(mv.x >> 16);
                // prefetch the parent's meta and legs (the next node of this walk in the common case)
                uint4 mu = make_uint4(0, 0, 0, 0);
                uint32_t h1 = 0, h2 = 0;
                if (v != 0) {
                    mu = sMETA[u];
                    h1 = sLG1[u * LT + l2.gl];
                    h2 = sLG2[u * LT + l2.gl];
                }
#ifdef FGR_TREE_TIMING
                nst++;
                nmul += nch >= 2;
                if (v == 0 && lane == 0 && m > 800)
                    printf("ROOT m=%d steps=%d multi=%d cycles=%lld per_step=%lld multiB=%lld handoff=%lld\n", m, nst, nmul,
                           clock64() - tst, (clock64() - tst) / nst, tmb / max(nmb, 1), tho / nst);
#endif
                uint32_t B;
                uint32_t Ev;
                if (nch >= 2 || v == 0) {
#ifdef FGR_TREE_TIMING
                    const long long q0 = clock64();
#endif
                    B = tree_multi_B<LT, NT, CAP>(g, sm, l2, v, prev, X, scrW, s_root);
#ifdef FGR_TREE_TIMING
                    tmb += clock64() - q0;
                    nmb++;
#endif
                    if (v == 0) break;   // the root's value and span are in s_root
                } else {
                    // at most one child (prev): B(ls) = min_l X(l) + max(vp[b], vp[l]) - min(vp[a], vp[l])
                    const uint32_t vpa = min(l2.myvp, mv.z), vpb = max(l2.myvp, mv.w);
                    const bool leaf = nch == 0;
                    uint32_t b0 = 0xFFFFFFFFu, b1 = 0xFFFFFFFFu, b2 = 0xFFFFFFFFu;
#pragma unroll
                    for (int l = 0; l < LT; l++) {
                        const uint32_t vl = g.viapre[l];
                        const uint32_t w = max(vpb, vl) - min(vpa, vl);
                        const uint32_t x = leaf ? 0u : X[l];
                        if (l % 3 == 0) b0 = __viaddmin_u32(x, w, b0);
                        else if (l % 3 == 1) b1 = __viaddmin_u32(x, w, b1);
                        else b2 = __viaddmin_u32(x, w, b2);
                    }
                    B = min(min(b0, b1), min(b2, FGR_INF));
                }
                // edge step: E_v(lt), lane = lt
                const int et = (int)(mv.y >> 16);
                if (et == TE_BENT) {
                    const uint32_t bp = sat_add(B, g1);
                    uint32_t e0 = 0xFFFFFFFFu, e1 = 0xFFFFFFFFu, e2 = 0xFFFFFFFFu;
#pragma unroll
                    for (int ls = 0; ls < LT; ls++) {
                        const uint32_t x = __shfl_sync(0xffffffffu, bp, ls);
                        if (ls % 3 == 0) e0 = __viaddmin_u32(x, l2.D[ls], e0);
                        else if (ls % 3 == 1) e1 = __viaddmin_u32(x, l2.D[ls], e1);
                        else e2 = __viaddmin_u32(x, l2.D[ls], e2);
                    }
                    Ev = sat_add(min(min(e0, e1), min(e2, FGR_INF)), g2);
                } else if (et == TE_HYB) {
                    const uint32_t* M = hyb_row<LT>(hy, a0 + v, l2.gl);
                    uint32_t e0 = FGR_INF;
#pragma unroll
                    for (int ls = 0; ls < LT; ls++) {
                        const uint32_t x = __shfl_sync(0xffffffffu, B, ls);
                        e0 = min(e0, sat_add(x, __ldg(M + ls)));
                    }
                    Ev = e0;
                } else {
                    Ev = sat_add(B, g1);   // straight edge (R7)
                }
#ifdef FGR_TREE_TIMING
                const long long q1 = clock64();
#endif
                if (lane < LT) sE[v * LT + lane] = Ev;
#pragma unroll
                for (int l = 0; l < LT; l++) X[l] = __shfl_sync(0xffffffffu, Ev, l);
                if (l2.gl == nbuf) myid = v;
                nbuf++;
                int next = u;
                if ((mu.x >> 16) != 1u) {   // several children: the last one to finish continues
                    __syncwarp();
                    int last = 0;
                    if (lane == 0) last = atom_dec_acqrel(&sPEND[u]) == 1u;
                    last = __shfl_sync(0xffffffffu, last, 0);
                    if (!last) next = -1;
                }
#ifdef FGR_TREE_TIMING
                tho += clock64() - q1;
#endif
                if (nbuf == LT || next < 0) {   // publish finished nodes to the P3 queue (one fence per batch)
                    __syncwarp();
                    int s0 = 0;
                    if (lane == 0) {
                        fence_acqrel_cta();
                        s0 = atomicAdd(&s_qtail, nbuf);
                    }
                    s0 = __shfl_sync(0xffffffffu, s0, 0);
                    if (lane < nbuf) reinterpret_cast<volatile uint16_t*>(sQ)[s0 + lane] = (uint16_t)myid;
                    nbuf = 0;
                }
                prev = v;
                cur = next;
                mv = mu;
                g1 = h1;
                g2 = h2;
            }
            if (nbuf > 0) {   // the root walk's last nodes
                __syncwarp();
                int s0 = 0;
                if (lane == 0) {
                    fence_acqrel_cta();
                    s0 = atomicAdd(&s_qtail, nbuf);
                }
                s0 = __shfl_sync(0xffffffffu, s0, 0);
                if (lane < nbuf) reinterpret_cast<volatile uint16_t*>(sQ)[s0 + lane] = (uint16_t)myid;
                nbuf = 0;
            }
            // no forward work left in this warp: argmin tables of finished nodes, GPW at a time
            while (true) {
                int base = 0;
                if (lane == 0) base = atomicAdd(&s_qhead, GPW);
                base = __shfl_sync(0xffffffffu, base, 0);
                if (base >= m - 1) break;
                if (glane && base + gi < m - 1) {
                    const volatile uint16_t* q = reinterpret_cast<const volatile uint16_t*>(sQ) + base + gi;
                    int v = *q;
                    while (v == 0xFFFF) { __nanosleep(64); v = *q; }
                    fence_acqrel_cta();
                    tree_node_argmin<LT, NT, CAP>(g, hy, sm, ln, v, a0, scrF);
#ifdef FGR_TREE_TIMING
                    if (ln.gl == 0) atomicAdd(&s_p3done, 1);
#endif
                }
                __syncwarp();
            }
        }
#ifdef FGR_TREE_TIMING
        __syncwarp();
        if (lane == 0) s_wt[0][warp] = clock64();
#endif
        cta_sync();
#ifdef FGR_TREE_TIMING
        if (lane == 0) s_wt[1][warp] = tclock();
        if (lane == 0 && *(volatile int*)&s_p3done != m - 1) atomicAdd(&s_viol, 1);
        cta_sync();
        if (tid == 0 && s_viol) printf("VIOLATION m=%d warps=%d\n", m, s_viol);
#endif
        TMARK(3);
        TMARK(4);
        // ---- P4: top-down backtrack (S5) along heavy paths, shallowest light depth first
#ifdef FGR_TREE_TIMING
        long long trd[6] = {0, 0, 0, 0, 0, 0};
        int trl[6] = {0, 0, 0, 0, 0, 0}, trn[6] = {0, 0, 0, 0, 0, 0};
#endif
        for (int r = 0; r < nr; r++) {
            const int q0 = s_rb[r], q1 = r > 0 ? s_rb[r - 1] : np;
#ifdef FGR_TREE_TIMING
            const long long t0r = tclock();
            if (tid == 0 && r < 6) {
                int mx = 0;
                for (int q = q0; q < q1; q++) mx = max(mx, (int)sPO[q + 1] - (int)sPO[q]);
                trl[r] = mx; trn[r] = q1 - q0;
            }
#endif
            for (int q = q0 + tid; q < q1; q += NT) {
                const int kb = sPO[q], ke = sPO[q + 1];
                int k = ke - 1;
                int v = sPN[k];
                int s;
                if (v == 0) s = (int)s_root[0];
                else { s = sPHI[v * NS + sSPAN[sPAR[v]]]; sSPAN[v] = (uint8_t)s; }
                if (v == 0) sSPAN[0] = (uint8_t)s;
                for (k = ke - 2; k >= kb; k -= 8) {   // node ids first, then the chain of phi lookups
                    int w[8];
#pragma unroll
                    for (int j = 0; j < 8; j++) w[j] = k - j >= kb ? (int)sPN[k - j] : -1;
#pragma unroll
                    for (int j = 0; j < 8; j++)
                        if (w[j] >= 0) { s = sPHI[w[j] * NS + s]; sSPAN[w[j]] = (uint8_t)s; }
                }
            }
            cta_sync();
#ifdef FGR_TREE_TIMING
            if (r < 6) trd[r] = tclock() - t0r;
#endif
        }
        TMARK(5);
#ifdef FGR_TREE_TIMING
        if (tid == 0 && m > 1000)
            printf("BACK m=%d r0 %lld/%d/%d r1 %lld/%d/%d r2 %lld/%d/%d r3 %lld/%d/%d r4 %lld/%d/%d\n", m, trd[0], trl[0], trn[0],
                   trd[1], trl[1], trn[1], trd[2], trl[2], trn[2], trd[3], trl[3], trn[3], trd[4], trl[4], trn[4]);
#endif
        // ---- P5: outputs; the S6 commit follows in k_commit_nets
        for (int i = 1 + tid; i < m; i += NT) {
            const int su = sSPAN[sPAR[i]];
            const int lo = s_tlo[su], hi = s_thi[su];
            const uint32_t* Ei = sE + i * LT;
            uint32_t be = Ei[lo];
            int lt = lo;
            for (int l = lo + 1; l <= hi; l++) {
                const uint32_t e = Ei[l];
                if (e < be) { be = e; lt = l; }
            }
            const int ls = sRECE[i * LT + lt];
            const int et = sET[i];
            const bool straight = et == TE_SH || et == TE_SV;
            const uint32_t bend = seg_bend(((hmask >> ls) & 1u) ? 0 : 1, ((hmask >> lt) & 1u) ? 0 : 1, straight);
            const uint32_t s = bend | ((uint32_t)ls << 8) | ((uint32_t)lt << 16) | ((uint32_t)straight << 24);
            if (o.rec_seg) o.rec_seg[o.rec_off[o.list_base + idx] + i] = s;
            else o.seg[a0 + i] = s;
        }
        if (tid == 0) {
            if (o.rec_seg) { o.rec_seg[o.rec_off[o.list_base + idx]] = 0xFFFFFFFFu; o.rec_cost[o.list_base + idx] = s_root[1]; }
            else { o.seg[a0] = 0xFFFFFFFFu; o.cost[net] = s_root[1]; }
        }
        cta_sync();
        TMARK(6);
#ifdef FGR_TREE_TIMING
        if (threadIdx.x == 0 && m > 400) {
            long long p2a = 1LL << 62, p2b = 0, qa = 1LL << 62, qb = 0;
            for (int w = 0; w < NT / 32; w++) {
                p2a = min(p2a, s_wt[0][w] - tmk[2]); p2b = max(p2b, s_wt[0][w] - tmk[2]);
                qa = min(qa, s_wt[1][w] - tmk[2]); qb = max(qb, s_wt[1][w] - tmk[2]);
            }
            printf("BAR m=%d pre=%lld..%lld post=%lld..%lld t3=%lld\n", m, p2a, p2b, qa, qb, tmk[3] - tmk[2]);
            printf("TREE m=%d np=%d nr=%d NT=%d load=%lld gather=%lld values=%lld argmin=%lld back=%lld out=%lld total=%lld "
                   "p23w=%lld..%lld\n",
                   m, np, nr, NT, tmk[1] - tmk[0], tmk[2] - tmk[1], tmk[3] - tmk[2], tmk[4] - tmk[3], tmk[5] - tmk[4],
                   tmk[6] - tmk[5], tmk[6] - tmk[0], p2a, p2b);
        }
#endif
    }
}

// P1 for the tree-kernel nets above 512 nodes, done by many SMs: every edge's leg costs, one task
// per thread (4 tasks per edge as in the kernel's own tables: 0 leg 1 H on row y_v, 1 leg 1 V on
// col x_v, 2 leg 2 V on col x_u, 3 leg 2 H on row y_u), written as rows LG1 [maxm][LT] | LG2
// [maxm][LT] per net, so that a lone large net does not pull its ~4000 prefix gathers through one
// SM.  Straight edges get INF on the layers of the other direction (R6, R7); hybrid edges use
// their transfer matrices instead.
template <int LT>
__global__ void __launch_bounds__(256) k_tree_legs(GridView g, NetsView nv, const int32_t* __restrict__ list, int count,
                                                   int chunks, int maxm, uint32_t* __restrict__ out, HybView hy) {
    pdl_trigger();   // the tree kernel may start its topology prologue
    pdl_wait();      // the refresh must be complete
    const int idx = blockIdx.x / chunks;
    if (idx >= count) return;
    const int net = list[idx];
    const int a0 = nv.off[net], m = nv.off[net + 1] - a0;
    const int task = (blockIdx.x % chunks) * 256 + threadIdx.x;
    if (task >= 4 * (m - 1)) return;
    const int hnet = hy.net ? hy.net[net] : -1;
    uint32_t* const L1 = out + (size_t)idx * 2 * maxm * LT;
    uint32_t* const L2 = L1 + (size_t)maxm * LT;
    const int v = 1 + (task >> 2), type = task & 3;
    const int u = nv.par[a0 + v];
    const int xv = nv.x[a0 + v], yv = nv.y[a0 + v], xu = nv.x[a0 + u], yu = nv.y[a0 + u];
    const int et = (yv == yu) ? TE_SH : (xv == xu) ? TE_SV : ((hnet >= 0 && hy.slot[a0 + v] >= 0) ? TE_HYB : TE_BENT);
    if (et == TE_HYB || (et == TE_SH && type != 0) || (et == TE_SV && type != 1)) return;
    const bool H = type == 0 || type == 3;
    const int line = type == 0 ? yv : type == 1 ? xv : type == 2 ? xu : yu;
    const int pa = H ? min(xv, xu) : min(yv, yu);
    const int pb = H ? max(xv, xu) : max(yv, yu);
    const uint32_t* P = H ? g.h.P : g.v.P;
    const uint32_t* SB = H ? g.h.SB : g.v.SB;
    const int len = H ? g.h.len : g.v.len, W = H ? g.h.W : g.v.W, nseg = H ? g.h.nseg : g.v.nseg;
    const int cnt = H ? g.h.cnt : g.v.cnt;
    uint32_t* dst = (type >= 2 ? L2 : L1) + (size_t)v * LT;
    const uint8_t* los = g.layer_of_slot[H ? 0 : 1];
    if (et != TE_BENT) {   // straight: the other direction's layers are impossible
        const uint8_t* lo2 = g.layer_of_slot[H ? 1 : 0];
        const int c2 = H ? g.v.cnt : g.h.cnt;
        for (int k2 = 0; k2 < c2; k2++) dst[lo2[k2]] = FGR_INF;
    }
    const size_t ia = ((size_t)line * len + pa) * W, ib = ((size_t)line * len + pb) * W;
    const size_t sa = ((size_t)line * nseg + (pa >> FGR_SEG_SHIFT)) * W;
    const size_t sb = ((size_t)line * nseg + (pb >> FGR_SEG_SHIFT)) * W;
    const bool oneseg = (pa >> FGR_SEG_SHIFT) == (pb >> FGR_SEG_SHIFT);   // segment bases cancel
    for (int q = 0; q < (W >> 2); q++) {
        const uint4 Pa = __ldg(reinterpret_cast<const uint4*>(P + ia) + q);
        const uint4 Pb = __ldg(reinterpret_cast<const uint4*>(P + ib) + q);
        uint4 Sa = make_uint4(0, 0, 0, 0), Sb = make_uint4(0, 0, 0, 0);
        if (!oneseg) {
            Sa = __ldg(reinterpret_cast<const uint4*>(SB + sa) + q);
            Sb = __ldg(reinterpret_cast<const uint4*>(SB + sb) + q);
        }
        if (4 * q + 0 < cnt) dst[los[4 * q + 0]] = (Sb.x + Pb.x) - (Sa.x + Pa.x);
        if (4 * q + 1 < cnt) dst[los[4 * q + 1]] = (Sb.y + Pb.y) - (Sa.y + Pa.y);
        if (4 * q + 2 < cnt) dst[los[4 * q + 2]] = (Sb.z + Pb.z) - (Sa.z + Pa.z);
        if (4 * q + 3 < cnt) dst[los[4 * q + 3]] = (Sb.w + Pb.w) - (Sa.w + Pa.w);
    }
}

// S6 for the nets of a tree-kernel launch: one thread per tree edge, blocks of 256 edges.
__global__ void __launch_bounds__(256) k_commit_nets(GridView g, NetsView nv, const int32_t* __restrict__ list, int count,
                                                     int chunks, Out o, HybView hy) {
    __shared__ Hdr hs;
    init_hdr(&hs, g);
    __syncthreads();
    const int idx = blockIdx.x / chunks;
    if (idx >= count) return;
    const int net = list[idx];
    const int a0 = nv.off[net], m = nv.off[net + 1] - a0;
    const int i = 1 + (blockIdx.x % chunks) * 256 + threadIdx.x;
    if (i >= m) return;
    const uint32_t s = o.rec_seg ? o.rec_seg[o.rec_off[o.list_base + idx] + i] : o.seg[a0 + i];
    const int u = nv.par[a0 + i];
    commit_edge(g, &hs, nv.x[a0 + i], nv.y[a0 + i], nv.x[a0 + u], nv.y[a0 + u], s, hyb_z(hy, a0 + i, s, g.L));
}

template <int LT, int NT, int CAP>
int tree_grid(const fgr_grid* g, int n) {
    using T = TL<LT, NT, CAP>;
    int per_sm = NT >= 384 ? 1 : (NT >= 256 ? 2 : 4);
    const int by_smem = g->max_smem / (T::BYTES + 2048);
    if (by_smem < per_sm) per_sm = by_smem < 1 ? 1 : by_smem;
    return n < per_sm * g->num_sms ? n : per_sm * g->num_sms;
}

template <int LT, int NT, int CAP>
cudaError_t launch_tree_v(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, const Out& o,
                          const HldPrep& hp, const uint32_t* legs, int legs_maxm) {
    using T = TL<LT, NT, CAP>;
    static int configured = 0;
    if (!configured) {
        cudaError_t e = cudaFuncSetAttribute(k_dp_tree<LT, NT, CAP>, cudaFuncAttributeMaxDynamicSharedMemorySize, T::BYTES);
        if (e != cudaSuccess) return e;
        configured = 1;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(tree_grid<LT, NT, CAP>(g, n));
    cfg.blockDim = dim3(NT);
    cfg.dynamicSmemBytes = T::BYTES;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k_dp_tree<LT, NT, CAP>, g->view, nv, list, n, o, hp, g->hy.view(), legs, legs_maxm);
}

template <int LT>
cudaError_t launch_tree_lt(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                           const Out& o, const HldPrep& hp, const uint32_t* legs, int legs_maxm) {
    if (maxm <= 128) return launch_tree_v<LT, 256, 128>(g, st, nv, list, n, o, hp, legs, legs_maxm);
    if (maxm <= 512) return launch_tree_v<LT, 384, 512>(g, st, nv, list, n, o, hp, legs, legs_maxm);
    return launch_tree_v<LT, kTreeBigNT, tree_cap512(LT)>(g, st, nv, list, n, o, hp, legs, legs_maxm);
}

template <int LT>
cudaError_t launch_legs_lt(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                           uint32_t* legs) {
    const int chunks = (4 * (maxm - 1) + 255) / 256;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(n * chunks));
    cfg.blockDim = dim3(256);
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k_tree_legs<LT>, g->view, nv, list, n, chunks, maxm, legs, g->hy.view());
}

}  // namespace

int fgr_tree_cap(const fgr_grid* g) {
    switch (g->L) {
#define FGR_LT(k) case k: return tree_cap512(k);
        FGR_LT(2) FGR_LT(3) FGR_LT(4) FGR_LT(5) FGR_LT(6) FGR_LT(7) FGR_LT(8) FGR_LT(9) FGR_LT(10) FGR_LT(11)
        FGR_LT(12) FGR_LT(13) FGR_LT(14) FGR_LT(15) FGR_LT(16)
#undef FGR_LT
        default: return 0;
    }
}

cudaError_t fgr_launch_tree_legs(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                                 uint32_t* legs) {
    if (n <= 0) return cudaSuccess;
    g->stats.kernel_launches++;
    switch (g->L) {
#define FGR_LT(k) case k: return launch_legs_lt<k>(g, st, nv, list, n, maxm, legs);
        FGR_LT(2) FGR_LT(3) FGR_LT(4) FGR_LT(5) FGR_LT(6) FGR_LT(7) FGR_LT(8) FGR_LT(9) FGR_LT(10) FGR_LT(11)
        FGR_LT(12) FGR_LT(13) FGR_LT(14) FGR_LT(15) FGR_LT(16)
#undef FGR_LT
        default: return cudaErrorInvalidValue;
    }
}

cudaError_t fgr_launch_tree(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                            const Out& o, bool commit, const HldPrep& hp, const uint32_t* legs, int legs_maxm) {
    if (n <= 0) return cudaSuccess;
    cudaError_t e;
    switch (g->L) {
#define FGR_LT(k) case k: e = launch_tree_lt<k>(g, st, nv, list, n, maxm, o, hp, legs, legs_maxm); break;
        FGR_LT(2) FGR_LT(3) FGR_LT(4) FGR_LT(5) FGR_LT(6) FGR_LT(7) FGR_LT(8) FGR_LT(9) FGR_LT(10) FGR_LT(11)
        FGR_LT(12) FGR_LT(13) FGR_LT(14) FGR_LT(15) FGR_LT(16)
#undef FGR_LT
        default: return cudaErrorInvalidValue;
    }
    if (e != cudaSuccess || !commit) return e;
    return fgr_launch_commit_nets(g, st, nv, list, n, maxm, o);
}

cudaError_t fgr_launch_commit_nets(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                                   const Out& o) {
    if (n <= 0 || maxm < 2) return cudaSuccess;
    g->stats.kernel_launches++;
    const int chunks = (maxm - 1 + 255) / 256;
    k_commit_nets<<<n * chunks, 256, 0, st>>>(g->view, nv, list, n, chunks, o, g->hy.view());
    return cudaGetLastError();
}
