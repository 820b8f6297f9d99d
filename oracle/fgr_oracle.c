/*
 * fgr_oracle.c — plain CPU oracle of FastGR's pattern-routing stage.
 *
 * TEST INFRASTRUCTURE ONLY (see fgr_oracle.h): tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs are the only users.  No
 * code is shared with the CUDA path.
 *
 * What it computes, in the order of SURVEY.md §8(c) "Algorithm (oracle)":
 *   1. cost table T_l[s] and edge cost ec = LEN + T_l[clamp(cap-dem,-S,S)]   (reading R1)
 *      via stack cost V(lo,hi) = sum_{k=lo}^{hi-1} VIA[k]                      (reading R2)
 *      wire cost of a leg = direct sum of ec over its unit edges (NO prefix sums)
 *   2. sort non-trivial nets by (HPWL over all nodes, net id)
 *   3. literal Algorithm 1 passes with an occupancy bitmap
 *   4. batches in sequence; each batch routed on the demand at its start,
 *      then committed (+1 per unit edge of every chosen leg)
 *   5. per-net tree DP: Eq. (1) path cost, Eq. (2) bottom-children cost (by
 *      span enumeration), Eq. (3) recurrence, generalised Eq. (4) root,
 *      then top-down backtrack
 *
 * Tie-breaks (reading R11): spans by (value, lo, hi); edge argmin by smallest
 * ls; child layer by smallest l.  Arithmetic: uint64 with an explicit INF for
 * "impossible" (a wire on a layer whose preferred direction does not match);
 * every finite result must be < 2^31 (ORC_RANGE otherwise).
 *
 * Parity status: pinned (tests/test_oracle_*.py: hand-worked W1-W4 and A-ex,
 * brute-force enumeration, invariants).  The cost *formula* itself (R1, R2) is
 * our reading of a passage that defers to another paper ("referring to the
 * cost scheme in [3]"): its similarity to FastGR/CUGR costs
 * is "parity unpinned".
 */
#include "fgr_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

#define INF ((uint64_t)1 << 62)
#define FINITE_LIMIT ((uint64_t)0x7FFFFFFF)

static uint64_t add(uint64_t a, uint64_t b) { return (a >= INF || b >= INF) ? INF : a + b; }

/* ---------------------------------------------------------------- costs */

/* T_l[s] = round_half_away(W_l / (1 + exp(slope * s))), s in [-S, S] (reading R1). */
int orc_cost_table(const orc_grid* g, int64_t* table) {
    int S = g->slack_clamp;
    for (int l = 0; l < g->nlayers; l++)
        for (int s = -S; s <= S; s++)
            table[(int64_t)l * (2 * S + 1) + (s + S)] =
                llround((double)g->ovf_weight[l] / (1.0 + exp(g->logistic_slope * (double)s)));
    return ORC_OK;
}

typedef struct {
    const orc_grid* g;
    const int32_t* demand;
    int64_t* table;
} cost_ctx;

static int32_t capacity_at(const orc_grid* g, int l, int y, int x) {
    if (g->edge_capacity) return g->edge_capacity[((int64_t)l * g->ny + y) * g->nx + x];
    return g->layer_capacity[l];
}

/* Cost of one unit wire edge on layer l stored at (y,x) of the dense layout. */
static uint64_t edge_cost(const cost_ctx* c, int l, int y, int x) {
    const orc_grid* g = c->g;
    int S = g->slack_clamp;
    int64_t slack = (int64_t)capacity_at(g, l, y, x) - c->demand[((int64_t)l * g->ny + y) * g->nx + x];
    if (slack < -S) slack = -S;
    if (slack > S) slack = S;
    return (uint64_t)g->len_cost + (uint64_t)c->table[(int64_t)l * (2 * S + 1) + (slack + S)];
}

/* cw: wire cost of the straight leg (xa,ya)-(xb,yb) on layer l.
 * Zero length -> 0.  Leg not along l's preferred direction -> INF (reading R6). */
static uint64_t wire_cost(const cost_ctx* c, int l, int xa, int ya, int xb, int yb) {
    if (xa == xb && ya == yb) return 0;
    if (ya == yb) {                                  /* horizontal leg */
        if (c->g->dir[l] != 0) return INF;
        int x0 = xa < xb ? xa : xb, x1 = xa < xb ? xb : xa;
        uint64_t s = 0;
        for (int x = x0; x < x1; x++) s += edge_cost(c, l, ya, x);
        return s;
    }
    if (xa == xb) {                                  /* vertical leg */
        if (c->g->dir[l] != 1) return INF;
        int y0 = ya < yb ? ya : yb, y1 = ya < yb ? yb : ya;
        uint64_t s = 0;
        for (int y = y0; y < y1; y++) s += edge_cost(c, l, y, xa);
        return s;
    }
    return INF;                                      /* not a straight leg */
}

/* cv: via stack between layers lo..hi at one G-cell (reading R2). */
static uint64_t via_stack(const orc_grid* g, int l1, int l2) {
    int lo = l1 < l2 ? l1 : l2, hi = l1 < l2 ? l2 : l1;
    uint64_t s = 0;
    for (int k = lo; k < hi; k++) s += (uint64_t)g->via_cost[k];
    return s;
}

/* ------------------------------------------------------------ validation */

int orc_validate(const orc_grid* g, const orc_nets* n, int32_t* bad_net) {
    for (int i = 0; i < n->num_nets; i++) {
        int a = n->node_offset[i], b = n->node_offset[i + 1];
        int bad = b <= a;
        for (int v = a; v < b && !bad; v++) {
            int loc = v - a;
            if (n->x[v] < 0 || n->x[v] >= g->nx || n->y[v] < 0 || n->y[v] >= g->ny) bad = 1;
            int lo = n->pin_lo[v], hi = n->pin_hi[v];
            if (!((lo == -1 && hi == -1) || (lo >= 0 && lo <= hi && hi < g->nlayers))) bad = 1;
            if (loc == 0) { if (n->parent[v] != -1) bad = 1; continue; }
            int p = n->parent[v];
            if (p < 0 || p >= loc) { bad = 1; continue; }
            if (n->x[a + p] == n->x[v] && n->y[a + p] == n->y[v]) bad = 1;  /* zero-length edge */
        }
        if (bad) { if (bad_net) *bad_net = i; return ORC_INVALID; }
    }
    return ORC_OK;
}

/* ------------------------------------------------------- Algorithm 1 */

typedef struct { int64_t key; int32_t id; } keyed;

static int cmp_keyed(const void* a, const void* b) {
    const keyed* x = (const keyed*)a; const keyed* y = (const keyed*)b;
    if (x->key != y->key) return x->key < y->key ? -1 : 1;
    return x->id < y->id ? -1 : (x->id > y->id);
}

static void net_bbox(const orc_nets* n, int i, int* x0, int* y0, int* x1, int* y1) {
    int a = n->node_offset[i], b = n->node_offset[i + 1];
    *x0 = *x1 = n->x[a]; *y0 = *y1 = n->y[a];
    for (int v = a; v < b; v++) {           /* bbox over ALL tree nodes (reading R14) */
        if (n->x[v] < *x0) *x0 = n->x[v];
        if (n->x[v] > *x1) *x1 = n->x[v];
        if (n->y[v] < *y0) *y0 = n->y[v];
        if (n->y[v] > *y1) *y1 = n->y[v];
    }
}

/*
 * Sort by ascending HPWL, ties by net id (reading R12),
 * then repeat Algorithm 1 until no nets remain
 * (PAPER.md L487-494).  "No conflict" = closed bounding boxes share no G-cell
 * (reading R13), tested literally with an occupancy bitmap of the batch.
 * Single-node nets are trivial: batch -1.
 */
int orc_plan(const orc_grid* g, const orc_nets* n, int32_t* batch_of_net, int32_t* num_batches) {
    int32_t bad;
    if (orc_validate(g, n, &bad) != ORC_OK) return ORC_INVALID;
    int N = n->num_nets;
    keyed* nets = (keyed*)malloc(sizeof(keyed) * (N > 0 ? N : 1));
    int R = 0;
    for (int i = 0; i < N; i++) {
        batch_of_net[i] = -1;
        if (n->node_offset[i + 1] - n->node_offset[i] < 2) continue;
        int x0, y0, x1, y1;
        net_bbox(n, i, &x0, &y0, &x1, &y1);
        nets[R].key = (int64_t)(x1 - x0) + (y1 - y0);
        nets[R].id = i;
        R++;
    }
    qsort(nets, R, sizeof(keyed), cmp_keyed);
    uint8_t* occ = (uint8_t*)calloc((size_t)g->nx * g->ny, 1);
    int b = 0;
    while (R > 0) {
        memset(occ, 0, (size_t)g->nx * g->ny);
        int keep = 0;
        for (int r = 0; r < R; r++) {           /* lines 3-8: scan the remaining nets in order */
            int x0, y0, x1, y1;
            net_bbox(n, nets[r].id, &x0, &y0, &x1, &y1);
            int conflict = 0;
            for (int y = y0; y <= y1 && !conflict; y++)
                for (int x = x0; x <= x1; x++)
                    if (occ[(int64_t)y * g->nx + x]) { conflict = 1; break; }
            if (!conflict) {                    /* push into batch, remove from nets */
                batch_of_net[nets[r].id] = b;
                for (int y = y0; y <= y1; y++)
                    for (int x = x0; x <= x1; x++) occ[(int64_t)y * g->nx + x] = 1;
            } else {
                nets[keep++] = nets[r];
            }
        }
        R = keep;
        b++;
    }
    *num_batches = b;
    free(occ);
    free(nets);
    return ORC_OK;
}

/* ------------------------------------------------------ tree DP per net */

/*
 * One net.  Node v != root owns the two-pin net v -> parent(v) ("Ps -> Pt" with
 * Ps = v the child/source side, Pt = u the parent/target side).
 *
 *   E[v][lt] = c*(Ps,Pt,lt)                      Eq. (3)
 *   B[v][ls] = cbc(Ps,ls)                        Eq. (2), by span enumeration
 *   F_v(lo,hi) = V(lo,hi) + sum_c min_{l in [lo,hi]} E[c][l]
 *   B[v][ls]   = min over spans [lo,hi] containing ls and the pin span of F_v
 *   root total = min over spans containing the root pin span of F_r   (generalised Eq. (4))
 */
/* Hybrid selection (reading R23): a bent tree edge whose
 * two-pin HPWL |dx|+|dy| lies in [hybrid_lo, hybrid_hi] is a "medium" two-pin
 * net and takes the hybrid L+Z patterns; every other edge takes the L patterns. */
static int is_hybrid_edge(const orc_pattern* pat, int xv, int yv, int xu, int yu) {
    if (!pat || xv == xu || yv == yu) return 0;
    int h = abs(xv - xu) + abs(yv - yu);
    return h >= pat->hybrid_lo && h <= pat->hybrid_hi;
}

/*
 * c*(Ps,Pt,lt) of one hybrid edge, §III-E/F (Eqs. (8)-(14), L831-1041,
 * and the hybrid candidate set, L1043-1092): the candidates are the two L
 * shapes (the bend pairs whose target bend point coincides with Pt, L1062-1068)
 * and the Z shapes whose bend points lie strictly inside the box (reading R24):
 *   HVH: Bs = (xm, yv), Bt = (xm, yu) for every xm strictly between xv and xu,
 *   VHV: Bs = (xv, ym), Bt = (xu, ym) for every ym strictly between yv and yu.
 * Eq. (8): c = cw(Ps,Bs,ls) + cv(Bs,ls,lb) + cw(Bs,Bt,lb) + cv(Bt,lb,lt) + cw(Bt,Pt,lt),
 * Eq. (9)/(14): min over ls, lb of cbc(Ps,ls) + c; Eq. (10): min over the candidates.
 * Tie-break (reading R25): the first minimum in the order (ls, candidate, lb),
 * candidates = the L shape first, then Z shapes by increasing xm / ym.
 * Writes E[lt], recE[lt] = ls and recZ[lt] = xm|ym | lb << 16 for a Z (else -1).
 */
static void hybrid_edge(const cost_ctx* c, const uint64_t* Bv, int xv, int yv, int xu, int yu,
                        uint64_t* E, uint8_t* recE, int32_t* recZ) {
    const orc_grid* g = c->g;
    int L = g->nlayers;
    int nxm = abs(xu - xv) - 1, nym = abs(yu - yv) - 1;      /* interior bend positions */
    int xlo = xv < xu ? xv : xu, ylo = yv < yu ? yv : yu;
    /* wire costs of the three legs of every Z candidate on every layer, by direct sums */
    uint64_t* hw = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)(nxm > 0 ? nxm : 1) * L * 3);
    uint64_t* vw = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)(nym > 0 ? nym : 1) * L * 3);
    for (int i = 0; i < nxm; i++) {
        int xm = xlo + 1 + i;
        for (int l = 0; l < L; l++) {
            hw[((size_t)i * L + l) * 3 + 0] = wire_cost(c, l, xv, yv, xm, yv);   /* Ps -> Bs */
            hw[((size_t)i * L + l) * 3 + 1] = wire_cost(c, l, xm, yv, xm, yu);   /* Bs -> Bt */
            hw[((size_t)i * L + l) * 3 + 2] = wire_cost(c, l, xm, yu, xu, yu);   /* Bt -> Pt */
        }
    }
    for (int i = 0; i < nym; i++) {
        int ym = ylo + 1 + i;
        for (int l = 0; l < L; l++) {
            vw[((size_t)i * L + l) * 3 + 0] = wire_cost(c, l, xv, yv, xv, ym);
            vw[((size_t)i * L + l) * 3 + 1] = wire_cost(c, l, xv, ym, xu, ym);
            vw[((size_t)i * L + l) * 3 + 2] = wire_cost(c, l, xu, ym, xu, yu);
        }
    }
    for (int lt = 0; lt < L; lt++) {
        uint64_t best = INF; int bls = 0; int32_t bz = -1;
        for (int ls = 0; ls < L; ls++) {
            if (g->dir[ls] != g->dir[lt]) {
                /* the L shape: bend 0 = (xu, yv) when leg 1 is horizontal, bend 1 = (xv, yu) */
                int bx = g->dir[ls] == 0 ? xu : xv, by = g->dir[ls] == 0 ? yv : yu;
                uint64_t cost = add(add(add(Bv[ls], wire_cost(c, ls, xv, yv, bx, by)), via_stack(g, ls, lt)),
                                    wire_cost(c, lt, bx, by, xu, yu));
                if (cost < best) { best = cost; bls = ls; bz = -1; }
                continue;
            }
            int hvh = g->dir[ls] == 0;
            int nm = hvh ? nxm : nym;
            const uint64_t* w = hvh ? hw : vw;
            for (int i = 0; i < nm; i++)
                for (int lb = 0; lb < L; lb++) {
                    uint64_t cost = add(Bv[ls], w[((size_t)i * L + ls) * 3 + 0]);   /* Eq. (11) */
                    cost = add(cost, add(via_stack(g, ls, lb), w[((size_t)i * L + lb) * 3 + 1]));   /* Eq. (12) */
                    cost = add(cost, add(via_stack(g, lb, lt), w[((size_t)i * L + lt) * 3 + 2]));   /* Eq. (13) */
                    if (cost < best) {
                        best = cost; bls = ls;
                        bz = (int32_t)((hvh ? xlo : ylo) + 1 + i) | (int32_t)(lb << 16);
                    }
                }
        }
        E[lt] = best;
        recE[lt] = (uint8_t)bls;
        recZ[lt] = bz;
    }
    free(hw); free(vw);
}

static int route_net(const cost_ctx* cc, const orc_nets* n, int32_t net, uint32_t* seg, uint32_t* net_cost,
                     const orc_pattern* pat, int32_t* zmid) {
    const orc_grid* g = cc->g;
    const cost_ctx c = *cc;
    int a = n->node_offset[net], m = n->node_offset[net + 1] - a, L = g->nlayers;
    if (zmid) for (int v = a; v < a + m; v++) zmid[v] = -1;
    if (m < 2) { if (m == 1) seg[a] = 0xFFFFFFFFu; *net_cost = 0; return ORC_OK; }

    uint64_t* E = (uint64_t*)malloc(sizeof(uint64_t) * m * L);   /* c*(v -> parent, lt) */
    uint8_t* recE = (uint8_t*)malloc((size_t)m * L);             /* argmin ls of E[v][lt] */
    int32_t* recZ = (int32_t*)malloc(sizeof(int32_t) * (size_t)m * L);   /* hybrid: Z bend of E[v][lt] or -1 */
    uint8_t* recLo = (uint8_t*)malloc((size_t)m * L);            /* argmin span of B[v][ls] */
    uint8_t* recHi = (uint8_t*)malloc((size_t)m * L);
    uint64_t* F = (uint64_t*)malloc(sizeof(uint64_t) * L * L);
    uint64_t* Bv = (uint64_t*)malloc(sizeof(uint64_t) * L);
    int* nchild = (int*)calloc(m + 1, sizeof(int));
    int* child = (int*)malloc(sizeof(int) * m);
    int* spanLo = (int*)malloc(sizeof(int) * m);
    int* spanHi = (int*)malloc(sizeof(int) * m);
    /* child lists (CSR) */
    for (int v = 1; v < m; v++) nchild[n->parent[a + v] + 1]++;
    for (int v = 0; v < m; v++) nchild[v + 1] += nchild[v];
    int* fill = (int*)malloc(sizeof(int) * (m + 1));
    memcpy(fill, nchild, sizeof(int) * (m + 1));
    for (int v = 1; v < m; v++) child[fill[n->parent[a + v]]++] = v;
    free(fill);

    int rc = ORC_OK;
    /* Children first: parent[i] < i, so descending index is a post-order. */
    for (int v = m - 1; v >= 0; v--) {
        /* F_v(lo,hi) for every span: via stack over the span + each child's best layer inside it */
        for (int lo = 0; lo < L; lo++)
            for (int hi = lo; hi < L; hi++) {
                uint64_t f = via_stack(g, lo, hi);
                for (int k = nchild[v]; k < nchild[v + 1]; k++) {
                    int ch = child[k];
                    uint64_t best = INF;
                    for (int l = lo; l <= hi; l++)
                        if (E[(int64_t)ch * L + l] < best) best = E[(int64_t)ch * L + l];
                    f = add(f, best);
                }
                F[lo * L + hi] = f;
            }
        int plo = n->pin_lo[a + v], phi = n->pin_hi[a + v];
        if (v == 0) {
            /* root: min over spans containing the pin span (Steiner root: any span) */
            uint64_t best = INF; int blo = 0, bhi = 0;
            for (int lo = 0; lo < L; lo++)
                for (int hi = lo; hi < L; hi++) {
                    if (plo >= 0 && !(lo <= plo && hi >= phi)) continue;
                    if (F[lo * L + hi] < best) { best = F[lo * L + hi]; blo = lo; bhi = hi; }
                }
            if (best >= FINITE_LIMIT) { rc = ORC_RANGE; break; }
            *net_cost = (uint32_t)best;
            spanLo[0] = blo; spanHi[0] = bhi;
            break;
        }
        /* Eq. (2): B[v][ls] = min over spans [lo,hi] that contain ls and the pin span */
        for (int ls = 0; ls < L; ls++) {
            int need_lo = ls, need_hi = ls;
            if (plo >= 0) { if (plo < need_lo) need_lo = plo; if (phi > need_hi) need_hi = phi; }
            uint64_t best = INF; int blo = 0, bhi = 0;
            for (int lo = 0; lo < L; lo++)
                for (int hi = lo; hi < L; hi++) {
                    if (!(lo <= need_lo && hi >= need_hi)) continue;
                    if (F[lo * L + hi] < best) { best = F[lo * L + hi]; blo = lo; bhi = hi; }
                }
            Bv[ls] = best;
            recLo[(int64_t)v * L + ls] = (uint8_t)blo;
            recHi[(int64_t)v * L + ls] = (uint8_t)bhi;
        }
        /* Eqs. (1), (3): E[v][lt] = min over ls of [ c(P{Ps,B_ls,T_lt}) + cbc(Ps,ls) ] */
        int u = n->parent[a + v];
        int xv = n->x[a + v], yv = n->y[a + v], xu = n->x[a + u], yu = n->y[a + u];
        int straight = (xv == xu) || (yv == yu);
        for (int lt = 0; lt < L; lt++) recZ[(int64_t)v * L + lt] = -1;
        if (is_hybrid_edge(pat, xv, yv, xu, yu)) {
            hybrid_edge(&c, Bv, xv, yv, xu, yu, E + (int64_t)v * L, recE + (int64_t)v * L, recZ + (int64_t)v * L);
            continue;
        }
        for (int lt = 0; lt < L; lt++) {
            uint64_t best = INF; int bls = 0;
            if (straight) {
                /* reading R7: one candidate, ls = lt, one leg */
                best = add(Bv[lt], wire_cost(&c, lt, xv, yv, xu, yu));
                bls = lt;
            } else {
                for (int bend = 0; bend < 2; bend++) {
                    /* bend 0: B = (xu, yv) (leg 1 horizontal); bend 1: B = (xv, yu) (leg 1 vertical) */
                    int bx = bend == 0 ? xu : xv, by = bend == 0 ? yv : yu;
                    for (int ls = 0; ls < L; ls++) {
                        uint64_t cost = add(add(add(Bv[ls], wire_cost(&c, ls, xv, yv, bx, by)),
                                                via_stack(g, ls, lt)),
                                            wire_cost(&c, lt, bx, by, xu, yu));  /* Eq. (1) */
                        if (cost < best) { best = cost; bls = ls; }
                    }
                }
            }
            E[(int64_t)v * L + lt] = best;
            recE[(int64_t)v * L + lt] = (uint8_t)bls;
        }
    }
    if (rc == ORC_OK) {
        /* Backtrack top-down (ascending index visits parents before children). */
        seg[a] = 0xFFFFFFFFu;
        for (int v = 1; v < m; v++) {
            int u = n->parent[a + v];
            int lo = spanLo[u], hi = spanHi[u];
            int lt = lo;
            for (int l = lo; l <= hi; l++)
                if (E[(int64_t)v * L + l] < E[(int64_t)v * L + lt]) lt = l;
            int ls = recE[(int64_t)v * L + lt];
            int xv = n->x[a + v], yv = n->y[a + v], xu = n->x[a + u], yu = n->y[a + u];
            int straight = (xv == xu) || (yv == yu);
            int bend = straight ? 0 : (g->dir[lt] == 1 ? 0 : 1);
            int32_t z = recZ[(int64_t)v * L + lt];
            if (z >= 0) {   /* a Z shape (hybrid edges only): 2 = HVH, 3 = VHV */
                bend = g->dir[ls] == 0 ? 2 : 3;
                if (zmid) zmid[a + v] = z;
            }
            seg[a + v] = (uint32_t)bend | ((uint32_t)ls << 8) | ((uint32_t)lt << 16) | ((uint32_t)straight << 24);
            spanLo[v] = recLo[(int64_t)v * L + ls];
            spanHi[v] = recHi[(int64_t)v * L + ls];
        }
    }
    free(E); free(recE); free(recZ); free(recLo); free(recHi); free(F); free(Bv);
    free(nchild); free(child); free(spanLo); free(spanHi);
    return rc;
}

int orc_route_net_ex(const orc_grid* g, const orc_nets* n, int32_t net, const int32_t* demand,
                     uint32_t* seg, uint32_t* net_cost, const orc_pattern* pat, int32_t* zmid) {
    cost_ctx c;
    c.g = g; c.demand = demand;
    c.table = (int64_t*)malloc(sizeof(int64_t) * g->nlayers * (2 * g->slack_clamp + 1));
    orc_cost_table(g, c.table);
    int rc = route_net(&c, n, net, seg, net_cost, pat, zmid);
    free(c.table);
    return rc;
}

int orc_route_net(const orc_grid* g, const orc_nets* n, int32_t net, const int32_t* demand,
                  uint32_t* seg, uint32_t* net_cost) {
    return orc_route_net_ex(g, n, net, demand, seg, net_cost, NULL, NULL);
}

/* +1 track on every unit edge of a leg (reading R16); zero-length legs add nothing. */
static void commit_leg(const orc_grid* g, int l, int xa, int ya, int xb, int yb, int32_t* demand) {
    if (ya == yb) {
        int x0 = xa < xb ? xa : xb, x1 = xa < xb ? xb : xa;
        for (int x = x0; x < x1; x++) demand[((int64_t)l * g->ny + ya) * g->nx + x] += 1;
    } else {
        int y0 = ya < yb ? ya : yb, y1 = ya < yb ? yb : ya;
        for (int y = y0; y < y1; y++) demand[((int64_t)l * g->ny + y) * g->nx + xa] += 1;
    }
}

/* The straight legs of one chosen route v -> u as (layer, xa, ya, xb, yb); returns how many (1..3).
 * Z shapes (bend 2 = HVH, 3 = VHV) take their middle coordinate and lb from zmid. */
static int route_legs(uint32_t s, int32_t z, int xv, int yv, int xu, int yu, int legs[3][5]) {
    int bend = s & 0xFF, ls = (s >> 8) & 0xFF, lt = (s >> 16) & 0xFF, straight = (s >> 24) & 0xFF;
    if (straight) {
        int q[5] = {lt, xv, yv, xu, yu};
        memcpy(legs[0], q, sizeof(q));
        return 1;
    }
    if (bend >= 2) {
        int mid = z & 0xFFFF, lb = (z >> 16) & 0xFF;
        int bsx = bend == 2 ? mid : xv, bsy = bend == 2 ? yv : mid;   /* source bend point Bs */
        int btx = bend == 2 ? mid : xu, bty = bend == 2 ? yu : mid;   /* target bend point Bt */
        int q0[5] = {ls, xv, yv, bsx, bsy}, q1[5] = {lb, bsx, bsy, btx, bty}, q2[5] = {lt, btx, bty, xu, yu};
        memcpy(legs[0], q0, sizeof(q0)); memcpy(legs[1], q1, sizeof(q1)); memcpy(legs[2], q2, sizeof(q2));
        return 3;
    }
    int bx = bend == 0 ? xu : xv, by = bend == 0 ? yv : yu;
    int q0[5] = {ls, xv, yv, bx, by}, q1[5] = {lt, bx, by, xu, yu};
    memcpy(legs[0], q0, sizeof(q0)); memcpy(legs[1], q1, sizeof(q1));
    return 2;
}

int orc_commit_net_ex(const orc_grid* g, const orc_nets* n, int32_t net, const uint32_t* seg, const int32_t* zmid,
                      int32_t* demand) {
    int a = n->node_offset[net], m = n->node_offset[net + 1] - a;
    for (int v = 1; v < m; v++) {
        int u = n->parent[a + v];
        int legs[3][5];
        int k = route_legs(seg[a + v], zmid ? zmid[a + v] : -1, n->x[a + v], n->y[a + v], n->x[a + u], n->y[a + u], legs);
        for (int j = 0; j < k; j++) commit_leg(g, legs[j][0], legs[j][1], legs[j][2], legs[j][3], legs[j][4], demand);
    }
    return ORC_OK;
}

int orc_commit_net(const orc_grid* g, const orc_nets* n, int32_t net, const uint32_t* seg, int32_t* demand) {
    return orc_commit_net_ex(g, n, net, seg, NULL, demand);
}

/*
 * Independent re-costing of a chosen route (used by the invariant tests):
 * wires + the via stack at every bend point (one per L, two per Z) + at every
 * node the via stack over the hull of {pin span, departure layer ls, arrival
 * layers lt of the children}.
 */
int orc_recost_net_ex(const orc_grid* g, const orc_nets* n, int32_t net, const int32_t* demand,
                      const uint32_t* seg, const int32_t* zmid, uint64_t* cost) {
    int a = n->node_offset[net], m = n->node_offset[net + 1] - a, L = g->nlayers, S = g->slack_clamp;
    cost_ctx c; c.g = g; c.demand = demand;
    c.table = (int64_t*)malloc(sizeof(int64_t) * L * (2 * S + 1));
    orc_cost_table(g, c.table);
    int* hlo = (int*)malloc(sizeof(int) * m);
    int* hhi = (int*)malloc(sizeof(int) * m);
    for (int v = 0; v < m; v++) {
        hlo[v] = n->pin_lo[a + v] >= 0 ? n->pin_lo[a + v] : L;
        hhi[v] = n->pin_hi[a + v] >= 0 ? n->pin_hi[a + v] : -1;
    }
    uint64_t total = 0;
    for (int v = 1; v < m; v++) {
        uint32_t s = seg[a + v];
        int ls = (s >> 8) & 0xFF, lt = (s >> 16) & 0xFF;
        int u = n->parent[a + v];
        int legs[3][5];
        int k = route_legs(s, zmid ? zmid[a + v] : -1, n->x[a + v], n->y[a + v], n->x[a + u], n->y[a + u], legs);
        for (int j = 0; j < k; j++) {
            total = add(total, wire_cost(&c, legs[j][0], legs[j][1], legs[j][2], legs[j][3], legs[j][4]));
            if (j > 0) total = add(total, via_stack(g, legs[j - 1][0], legs[j][0]));   /* bend point vias */
        }
        if (ls < hlo[v]) hlo[v] = ls;
        if (ls > hhi[v]) hhi[v] = ls;
        if (lt < hlo[u]) hlo[u] = lt;
        if (lt > hhi[u]) hhi[u] = lt;
    }
    for (int v = 0; v < m; v++)
        if (hhi[v] >= hlo[v]) total = add(total, via_stack(g, hlo[v], hhi[v]));
    *cost = total;
    free(c.table); free(hlo); free(hhi);
    return ORC_OK;
}

int orc_recost_net(const orc_grid* g, const orc_nets* n, int32_t net, const int32_t* demand,
                   const uint32_t* seg, uint64_t* cost) {
    return orc_recost_net_ex(g, n, net, demand, seg, NULL, cost);
}

static uint64_t fnv1a(const int32_t* d, int64_t n) {
    uint64_t h = 1469598103934665603ULL;
    const uint8_t* p = (const uint8_t*)d;
    for (int64_t i = 0; i < n * 4; i++) { h ^= p[i]; h *= 1099511628211ULL; }
    return h;
}

/*
 * The stage: batches in sequence.  Batch-synchronous mode routes
 * every net of batch b on the demand at the start of b, then commits them all;
 * sequential mode commits after each net (identical by reading R13, checked by
 * a test).  batch_hash[b] = FNV-1a of the demand after batch b (diff bisection).
 */
int orc_route(const orc_grid* g, const orc_nets* n, const int32_t* batch_of_net, int32_t num_batches,
              int32_t* demand, uint32_t* seg, uint32_t* net_cost, int sequential_within_batch,
              uint64_t* batch_hash) {
    return orc_route_ex(g, n, batch_of_net, num_batches, demand, seg, net_cost, sequential_within_batch, batch_hash,
                        NULL, NULL);
}

int orc_route_ex(const orc_grid* g, const orc_nets* n, const int32_t* batch_of_net, int32_t num_batches,
                 int32_t* demand, uint32_t* seg, uint32_t* net_cost, int sequential_within_batch,
                 uint64_t* batch_hash, const orc_pattern* pat, int32_t* zmid) {
    int32_t bad;
    if (orc_validate(g, n, &bad) != ORC_OK) return ORC_INVALID;
    int N = n->num_nets;
    int64_t dsize = (int64_t)g->nlayers * g->ny * g->nx;
    /* bucket nets by batch, ascending id inside a batch */
    int* cnt = (int*)calloc(num_batches + 1, sizeof(int));
    for (int i = 0; i < N; i++) {
        if (batch_of_net[i] >= num_batches) { free(cnt); return ORC_INVALID; }
        if (batch_of_net[i] >= 0) cnt[batch_of_net[i] + 1]++;
        else {
            int a = n->node_offset[i];
            for (int v = a; v < n->node_offset[i + 1]; v++) { seg[v] = 0xFFFFFFFFu; if (zmid) zmid[v] = -1; }
            net_cost[i] = 0;
        }
    }
    for (int b = 0; b < num_batches; b++) cnt[b + 1] += cnt[b];
    int* lst = (int*)malloc(sizeof(int) * (N > 0 ? N : 1));
    int* pos = (int*)malloc(sizeof(int) * (num_batches + 1));
    memcpy(pos, cnt, sizeof(int) * (num_batches + 1));
    for (int i = 0; i < N; i++) if (batch_of_net[i] >= 0) lst[pos[batch_of_net[i]]++] = i;
    int rc = ORC_OK;
    cost_ctx c;
    c.g = g; c.demand = demand;
    c.table = (int64_t*)malloc(sizeof(int64_t) * g->nlayers * (2 * g->slack_clamp + 1));
    orc_cost_table(g, c.table);
    for (int b = 0; b < num_batches && rc == ORC_OK; b++) {
        for (int k = cnt[b]; k < cnt[b + 1] && rc == ORC_OK; k++) {
            rc = route_net(&c, n, lst[k], seg, &net_cost[lst[k]], pat, zmid);
            if (sequential_within_batch) orc_commit_net_ex(g, n, lst[k], seg, zmid, demand);
        }
        if (!sequential_within_batch)
            for (int k = cnt[b]; k < cnt[b + 1]; k++) orc_commit_net_ex(g, n, lst[k], seg, zmid, demand);
        if (batch_hash) batch_hash[b] = fnv1a(demand, dsize);
    }
    free(c.table); free(cnt); free(lst); free(pos);
    return rc;
}

/* ------------------------------------------- overflow extraction (NEXT #3) */

/*
 * Rip-up set after the pattern-routing stage (§III-A: "we first
 * extract the nets to rip up"; §III-G: "rewire the nets with violations").
 * Reading R26: a wire edge is overflowed when its demand exceeds its capacity; a net
 * is violating when one of its committed legs covers an overflowed edge.
 * totals[0] = overflowed wire edges, totals[1] = sum of (demand - capacity) over them.
 */
int orc_overflow(const orc_grid* g, const orc_nets* n, const uint32_t* seg, const int32_t* zmid,
                 const int32_t* demand, uint8_t* violating, int64_t* totals) {
    int L = g->nlayers;
    int64_t cnt = 0, sum = 0;
    for (int l = 0; l < L; l++)
        for (int y = 0; y < g->ny; y++)
            for (int x = 0; x < g->nx; x++) {
                if (g->dir[l] == 0 && x == g->nx - 1) continue;   /* no wire edge there */
                if (g->dir[l] == 1 && y == g->ny - 1) continue;
                int64_t over = (int64_t)demand[((int64_t)l * g->ny + y) * g->nx + x] - capacity_at(g, l, y, x);
                if (over > 0) { cnt++; sum += over; }
            }
    totals[0] = cnt;
    totals[1] = sum;
    for (int i = 0; i < n->num_nets; i++) {
        int a = n->node_offset[i], m = n->node_offset[i + 1] - a, bad = 0;
        for (int v = 1; v < m && !bad; v++) {
            int u = n->parent[a + v];
            int legs[3][5];
            int k = route_legs(seg[a + v], zmid ? zmid[a + v] : -1, n->x[a + v], n->y[a + v], n->x[a + u],
                               n->y[a + u], legs);
            for (int j = 0; j < k && !bad; j++) {
                int l = legs[j][0], xa = legs[j][1], ya = legs[j][2], xb = legs[j][3], yb = legs[j][4];
                if (ya == yb) {
                    for (int x = (xa < xb ? xa : xb); x < (xa < xb ? xb : xa); x++)
                        if (demand[((int64_t)l * g->ny + ya) * g->nx + x] > capacity_at(g, l, ya, x)) { bad = 1; break; }
                } else {
                    for (int y = (ya < yb ? ya : yb); y < (ya < yb ? yb : ya); y++)
                        if (demand[((int64_t)l * g->ny + y) * g->nx + xa] > capacity_at(g, l, y, xa)) { bad = 1; break; }
                }
            }
        }
        violating[i] = (uint8_t)bad;
    }
    return ORC_OK;
}

/*
 * Ordered task graph of a set of routing tasks (§III-B, Fig. 6):
 *   task IDs = the tasks sorted by (HPWL, net id) ("the task ID indicates the sorting
 *   result", L461-462; sort key as reading R12);
 *   conflict = closed bounding boxes share a G-cell (reading R13);
 *   root task batch = one pass of Algorithm 1 over the sorted tasks (L432-448);
 *   every conflicting pair is ordered root -> non-root (L454-456), else from the
 *   smaller task ID to the larger (L457-459).
 * Outputs: order[t] = net id of task t; is_root[t]; successors in CSR by task ID,
 * ascending.  ORC_RANGE (with *num_edges set) when the edges exceed `cap`.
 */
int orc_task_graph(const orc_grid* g, const orc_nets* n, const int32_t* tasks, int32_t count, int32_t* order,
                   uint8_t* is_root, int32_t* succ_off, int32_t* succ, int64_t cap, int64_t* num_edges) {
    keyed* t = (keyed*)malloc(sizeof(keyed) * (count > 0 ? count : 1));
    int* bx = (int*)malloc(sizeof(int) * 4 * (count > 0 ? count : 1));
    for (int i = 0; i < count; i++) {
        int x0, y0, x1, y1;
        net_bbox(n, tasks[i], &x0, &y0, &x1, &y1);
        t[i].key = (int64_t)(x1 - x0) + (y1 - y0);
        t[i].id = tasks[i];
    }
    qsort(t, count, sizeof(keyed), cmp_keyed);
    for (int i = 0; i < count; i++) {
        order[i] = t[i].id;
        net_bbox(n, t[i].id, &bx[4 * i], &bx[4 * i + 1], &bx[4 * i + 2], &bx[4 * i + 3]);
    }
    /* root batch: Algorithm 1 lines 1-8, literally (occupancy bitmap of the batch) */
    uint8_t* occ = (uint8_t*)calloc((size_t)g->nx * g->ny, 1);
    for (int i = 0; i < count; i++) {
        int conflict = 0;
        for (int y = bx[4 * i + 1]; y <= bx[4 * i + 3] && !conflict; y++)
            for (int x = bx[4 * i]; x <= bx[4 * i + 2]; x++)
                if (occ[(int64_t)y * g->nx + x]) { conflict = 1; break; }
        is_root[i] = (uint8_t)!conflict;
        if (!conflict)
            for (int y = bx[4 * i + 1]; y <= bx[4 * i + 3]; y++)
                for (int x = bx[4 * i]; x <= bx[4 * i + 2]; x++) occ[(int64_t)y * g->nx + x] = 1;
    }
    free(occ);
    /* every conflicting pair, oriented; CSR by source, successors ascending */
    int64_t ne = 0;
    for (int i = 0; i <= count; i++) succ_off[i] = 0;
    for (int pass = 0; pass < 2; pass++) {
        int64_t k = 0;
        for (int a = 0; a < count; a++) {
            if (pass == 1) succ_off[a] = (int32_t)k;
            for (int b = 0; b < count; b++) {
                if (a == b) continue;
                int touch = !(bx[4 * a + 2] < bx[4 * b] || bx[4 * b + 2] < bx[4 * a] ||
                              bx[4 * a + 3] < bx[4 * b + 1] || bx[4 * b + 3] < bx[4 * a + 1]);
                if (!touch) continue;
                int a_first = is_root[a] ? 1 : (is_root[b] ? 0 : a < b);
                if (!a_first) continue;                       /* the edge is b -> a */
                if (pass == 1 && k < cap) succ[k] = b;
                k++;
            }
        }
        if (pass == 1) succ_off[count] = (int32_t)k;
        ne = k;
    }
    *num_edges = ne;
    free(t); free(bx);
    return ne > cap ? ORC_RANGE : ORC_OK;
}
