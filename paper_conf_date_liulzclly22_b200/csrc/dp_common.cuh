// dp_common.cuh — device helpers shared by the tree-DP kernels (dp.cu, dp_walk.cu):
// per-block constants, route records, leg gathers, the S6 commit.  Internal, not ABI.
#pragma once
#include "fgr_internal.cuh"

namespace {

__host__ __device__ constexpr int groups_of(int LT) { return (32 / LT) < 4 ? (32 / LT) : 4; }
__host__ __device__ inline size_t a16(size_t b) { return (b + 15) & ~(size_t)15; }

struct Hdr {                  // per-block constants copied to shared memory
    uint32_t viapre[FGR_MAXL + 1];
    uint8_t dir[FGR_MAXL];
    uint8_t slot[FGR_MAXL];
    uint8_t zlo[FGR_MAXL];    // smallest lo with V(lo, a) == 0 (zero-cost via run below a)
};

__device__ inline void init_hdr(Hdr* h, const GridView& g) {
    for (int i = threadIdx.x; i <= FGR_MAXL; i += blockDim.x) h->viapre[i] = g.viapre[i];
    for (int i = threadIdx.x; i < FGR_MAXL; i += blockDim.x) {
        h->dir[i] = g.dir[i];
        h->slot[i] = g.slot[i];
        int z = i;
        while (z > 0 && g.viapre[z - 1] == g.viapre[i]) z--;
        h->zlo[i] = (uint8_t)z;
    }
}


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

// Bend field of a chosen route: 0/1 = the L shapes (bend 0 when lt is vertical); a
// departure and arrival layer of the same direction on a bent edge is a Z shape of a
// hybrid edge: 2 = HVH, 3 = VHV (§III-E).
__device__ __forceinline__ uint32_t seg_bend(int dls, int dlt, bool straight) {
    if (straight) return 0u;
    if (dls == dlt) return dls == 0 ? 2u : 3u;
    return dlt == 1 ? 0u : 1u;
}

// Z argmin (mid | lb << 16) of a chosen Z route of global node gv, or 0 for an L shape.
__device__ __forceinline__ uint32_t hyb_z(const HybView& hy, int gv, uint32_t seg, int L) {
    if ((seg & 0xFF) < 2 || !hy.net) return 0u;
    const int s = hy.slot[gv];
    const int ls = (seg >> 8) & 0xFF, lt = (seg >> 16) & 0xFF;
    return hy.A[((size_t)s * L + lt) * L + ls];
}

// S6: +1 on every unit edge of a leg (fire-and-forget RED), and mark the touched
// 32-position segments and their line stale for the next refresh (plain byte stores).
__device__ __forceinline__ void commit_leg(const GridView& g, const DirView& d, int line, int a, int b, int sl) {
    if (a >= b) return;
    int32_t* D = d.D + (size_t)line * d.len * d.W + sl;
    for (int p = a; p < b; p++) atomicAdd(D + (size_t)p * d.W, 1);
    const int s0 = a >> FGR_SEG_SHIFT, s1 = (b - 1) >> FGR_SEG_SHIFT;
    uint8_t* f = g.dseg + d.seg_base + (size_t)line * d.nseg;
    for (int s = s0; s <= s1; s++) f[s] = 1;
    g.dline[d.line_base + line] = 1;
}

__device__ __forceinline__ void commit_edge(const GridView& g, const Hdr* h, int xv, int yv, int xu, int yu, uint32_t seg,
                                            uint32_t z) {
    const int bend = seg & 0xFF, ls = (seg >> 8) & 0xFF, lt = (seg >> 16) & 0xFF, straight = (seg >> 24) & 0xFF;
    if (straight) {
        if (yv == yu) commit_leg(g, g.h, yv, min(xv, xu), max(xv, xu), h->slot[lt]);
        else commit_leg(g, g.v, xv, min(yv, yu), max(yv, yu), h->slot[lt]);
        return;
    }
    if (bend >= 2) {   // Z shape (hybrid edge): three legs through Bs and Bt, middle layer lb
        const int mid = (int)(z & 0xFFFF), lb = (int)((z >> 16) & 0xFF);
        if (bend == 2) {   // HVH: row y_v to xm (ls), column xm (lb), row y_u from xm (lt)
            commit_leg(g, g.h, yv, min(xv, mid), max(xv, mid), h->slot[ls]);
            commit_leg(g, g.v, mid, min(yv, yu), max(yv, yu), h->slot[lb]);
            commit_leg(g, g.h, yu, min(mid, xu), max(mid, xu), h->slot[lt]);
        } else {           // VHV: column x_v to ym (ls), row ym (lb), column x_u from ym (lt)
            commit_leg(g, g.v, xv, min(yv, mid), max(yv, mid), h->slot[ls]);
            commit_leg(g, g.h, mid, min(xv, xu), max(xv, xu), h->slot[lb]);
            commit_leg(g, g.v, xu, min(mid, yu), max(mid, yu), h->slot[lt]);
        }
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

// Flattened (group, item) iteration: item counts per group n[q]; returns the group of item `it`.
template <int G>
struct Flat {
    int pre[G + 1];
    __device__ __forceinline__ void build(const int (&n)[G]) {
        pre[0] = 0;
#pragma unroll
        for (int q = 0; q < G; q++) pre[q + 1] = pre[q] + n[q];
    }
    __device__ __forceinline__ int total() const { return pre[G]; }
    __device__ __forceinline__ int group(int it) const {
        int q = 0;
#pragma unroll
        for (int k = 1; k < G; k++) q += (it >= pre[k]) ? 1 : 0;
        return q;
    }
    __device__ __forceinline__ int base(int q) const {
        int b = 0;
#pragma unroll
        for (int k = 0; k < G; k++) b = (k == q) ? pre[k] : b;
        return b;
    }
};

}  // namespace
