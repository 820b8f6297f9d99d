/*
 * fgr_gen.c — seeded synthetic design generator (workload layer L0).
 *
 * This module is SHARED INPUT PLUMBING for both the CUDA path and the oracle.
 * It holds none of the method's arithmetic: no edge cost, no via cost, no DP,
 * no batching.  It only draws a grid (dims, directions, capacities) and nets
 * (pin points mapped to G-cells plus a given tree topology), following the
 * recipe in DESIGN.md §"Input recipe" (SURVEY.md §8(d) "Synthetic inputs").
 *
 * Paper passages the *shape* of the input follows:
 *   - nets are point sets {(x1,y1)..(xn,yn)} on the G-cell grid
 *   - pins are mapped to G-cells
 *   - multipin nets are given as a tree of two-pin nets
 *   - one preferred direction per layer
 *
 * Output net format (see include/fastgr.h, fgr_nets):
 *   node_offset[N+1] CSR; node 0 of each net is its root; parent[i] < i (net-local)
 *   x,y int16; pin_lo,pin_hi int8 (-1,-1 = Steiner / paper-literal node).
 *
 * RNG: splitmix64 seeding xoshiro256**; doubles via the top 53 bits.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

/* ------------------------------------------------------------------ RNG */
typedef struct { uint64_t s[4]; } rng_t;

static uint64_t splitmix64(uint64_t* x) {
    uint64_t z = (*x += 0x9E3779B97F4A7C15ULL);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}
static uint64_t rotl(uint64_t x, int k) { return (x << k) | (x >> (64 - k)); }
static uint64_t rng_next(rng_t* r) {
    uint64_t* s = r->s;
    uint64_t result = rotl(s[1] * 5, 7) * 9;
    uint64_t t = s[1] << 17;
    s[2] ^= s[0]; s[3] ^= s[1]; s[1] ^= s[2]; s[0] ^= s[3];
    s[2] ^= t; s[3] = rotl(s[3], 45);
    return result;
}
static void rng_seed(rng_t* r, uint64_t seed) {
    uint64_t x = seed;
    for (int i = 0; i < 4; i++) r->s[i] = splitmix64(&x);
}
static double rng_u01(rng_t* r) { return (double)(rng_next(r) >> 11) * (1.0 / 9007199254740992.0); }
/* integer uniform in [lo, hi] inclusive */
static int64_t rng_int(rng_t* r, int64_t lo, int64_t hi) {
    uint64_t span = (uint64_t)(hi - lo + 1);
    return lo + (int64_t)(rng_next(r) % span);
}
static double rng_normal(rng_t* r) {
    double u1 = rng_u01(r), u2 = rng_u01(r);
    if (u1 < 1e-300) u1 = 1e-300;
    return sqrt(-2.0 * log(u1)) * cos(6.283185307179586 * u2);
}

/* ------------------------------------------------------------ parameters */
typedef struct {
    int32_t nx, ny, nlayers;
    int32_t num_nets;
    uint64_t seed;
    int32_t layer_capacity[16];
    int32_t pin_dist;          /* 0 = ISPD-like heavy tail, 1 = uniform k in [kmin,kmax] */
    int32_t kmin, kmax;
    double  hpwl_sigma;        /* lognormal sigma (0.7) */
    double  hpwl_base;         /* median = hpwl_base + 2*sqrt(k)  (3.0) */
    double  literal_frac;      /* fraction of nets with no pin layers (paper-literal) */
    int32_t hotspots;          /* number of gaussian hotspots */
    double  hot_frac;          /* fraction of nets centred in hotspots */
    double  hot_sigma_frac;    /* hotspot sigma as fraction of min(nx,ny) */
    int32_t congested_core;    /* 1 = central 1/3 x 1/3 at 3x density and 0.5x capacity */
    int32_t steiner;           /* 1 = one pass of 3-terminal median Steiner insertion */
} gen_params;

typedef struct {
    int32_t nx, ny, nlayers;
    uint8_t dir[16];
    int32_t layer_capacity[16];
    uint8_t* edge_capacity;    /* [nlayers][ny][nx] or NULL */
    int32_t num_nets, num_nodes;
    int32_t* node_offset;
    int16_t *x, *y;
    int8_t *pin_lo, *pin_hi;
    int32_t* parent;
    int64_t cap_nodes;
} gen_design;

static void push_reserve(gen_design* d, int64_t need) {
    if (need <= d->cap_nodes) return;
    int64_t c = d->cap_nodes ? d->cap_nodes : 1024;
    while (c < need) c *= 2;
    d->x = (int16_t*)realloc(d->x, c * sizeof(int16_t));
    d->y = (int16_t*)realloc(d->y, c * sizeof(int16_t));
    d->pin_lo = (int8_t*)realloc(d->pin_lo, c);
    d->pin_hi = (int8_t*)realloc(d->pin_hi, c);
    d->parent = (int32_t*)realloc(d->parent, c * sizeof(int32_t));
    d->cap_nodes = c;
}

/* ISPD-like pin count distribution. */
static int draw_k(rng_t* r, const gen_params* p) {
    if (p->pin_dist == 1) return (int)rng_int(r, p->kmin, p->kmax);
    static const double prob[10] = {.52, .18, .09, .05, .04, .06, .04, .015, .004, .001};
    static const int lo[10] = {2, 3, 4, 5, 6, 7, 11, 21, 51, 201};
    static const int hi[10] = {2, 3, 4, 5, 6, 10, 20, 50, 200, 1000};
    double u = rng_u01(r), acc = 0;
    for (int i = 0; i < 10; i++) {
        acc += prob[i];
        if (u < acc || i == 9) return (int)rng_int(r, lo[i], hi[i]);
    }
    return 2;
}

typedef struct { int x, y, lo, hi; } node_t;

static int iabs(int a) { return a < 0 ? -a : a; }
static int med3(int a, int b, int c) {
    if (a > b) { int t = a; a = b; b = t; }
    if (b > c) { b = c; }
    return a > b ? a : b;
}

/*
 * Build one net: pins -> merged cells -> Prim MST rooted at node 0 -> optional
 * median Steiner pass -> DFS preorder renumbering (parent[i] < i).
 * Scratch arrays sized by caller.
 */
typedef struct {
    node_t* nodes; int* par; int* newidx; int* order; int* stack;
    int* dist; int* in; int cap;
    int* cell_mark; /* per-grid-cell last net id touching it (merge) */
    int* cell_node;
} scratch_t;

static void scratch_reserve(scratch_t* s, int k) {
    int need = 2 * k + 8;
    if (need <= s->cap) return;
    s->cap = need;
    s->nodes = (node_t*)realloc(s->nodes, need * sizeof(node_t));
    s->par = (int*)realloc(s->par, need * sizeof(int));
    s->newidx = (int*)realloc(s->newidx, need * sizeof(int));
    s->order = (int*)realloc(s->order, need * sizeof(int));
    s->stack = (int*)realloc(s->stack, need * sizeof(int));
    s->dist = (int*)realloc(s->dist, need * sizeof(int));
    s->in = (int*)realloc(s->in, need * sizeof(int));
}

static int has_node_at(const node_t* n, int m, int x, int y) {
    for (int i = 0; i < m; i++) if (n[i].x == x && n[i].y == y) return 1;
    return 0;
}

int fgr_gen_design(const gen_params* p, gen_design* out) {
    memset(out, 0, sizeof(*out));
    if (p->nx < 2 || p->ny < 2 || p->nlayers < 2 || p->nlayers > 16 || p->num_nets < 0) return 1;
    rng_t rng; rng_seed(&rng, p->seed);
    out->nx = p->nx; out->ny = p->ny; out->nlayers = p->nlayers;
    for (int l = 0; l < p->nlayers; l++) { out->dir[l] = (uint8_t)(l & 1); out->layer_capacity[l] = p->layer_capacity[l]; }
    int nx = p->nx, ny = p->ny, L = p->nlayers;
    int cx0 = nx / 3, cx1 = (2 * nx) / 3, cy0 = ny / 3, cy1 = (2 * ny) / 3;  /* core [cx0,cx1) x [cy0,cy1) */
    if (p->congested_core) {
        out->edge_capacity = (uint8_t*)malloc((size_t)L * nx * ny);
        for (int l = 0; l < L; l++)
            for (int y = 0; y < ny; y++)
                for (int x = 0; x < nx; x++) {
                    int c = p->layer_capacity[l];
                    if (x >= cx0 && x < cx1 && y >= cy0 && y < cy1) c = c / 2;
                    if (c > 255) c = 255;
                    out->edge_capacity[((size_t)l * ny + y) * nx + x] = (uint8_t)c;
                }
    }
    /* hotspot centres */
    double hx[64], hy[64];
    int H = p->hotspots > 64 ? 64 : p->hotspots;
    for (int i = 0; i < H; i++) { hx[i] = rng_u01(&rng) * nx; hy[i] = rng_u01(&rng) * ny; }
    double hsig = p->hot_sigma_frac * (nx < ny ? nx : ny);

    out->num_nets = p->num_nets;
    out->node_offset = (int32_t*)malloc(((size_t)p->num_nets + 1) * sizeof(int32_t));
    scratch_t s; memset(&s, 0, sizeof(s));
    int64_t M = 0;
    out->node_offset[0] = 0;
    for (int n = 0; n < p->num_nets; n++) {
        int k = draw_k(&rng, p);
        int literal = rng_u01(&rng) < p->literal_frac;
        /* centre */
        double cx, cy;
        double u = rng_u01(&rng);
        if (p->congested_core) {
            if (u < 3.0 / 11.0) { cx = cx0 + rng_u01(&rng) * (cx1 - cx0); cy = cy0 + rng_u01(&rng) * (cy1 - cy0); }
            else {
                do { cx = rng_u01(&rng) * nx; cy = rng_u01(&rng) * ny; }
                while (cx >= cx0 && cx < cx1 && cy >= cy0 && cy < cy1);
            }
        } else if (H > 0 && u < p->hot_frac) {
            int h = (int)rng_int(&rng, 0, H - 1);
            do {   /* resample points that fall off the chip (no pile-up on the border) */
                cx = hx[h] + hsig * rng_normal(&rng); cy = hy[h] + hsig * rng_normal(&rng);
            } while (cx < 0 || cx >= nx || cy < 0 || cy >= ny);
        } else { cx = rng_u01(&rng) * nx; cy = rng_u01(&rng) * ny; }
        /* size */
        double med = p->hpwl_base + 2.0 * sqrt((double)k);
        int h = (int)llround(exp(log(med) + p->hpwl_sigma * rng_normal(&rng)));
        if (h < 1) h = 1;
        if (h > nx + ny - 2) h = nx + ny - 2;
        int w = (int)llround(h * (0.25 + 0.5 * rng_u01(&rng)));
        int hh = h - w;
        if (w > nx - 1) { w = nx - 1; }
        if (hh > ny - 1) { hh = ny - 1; }
        int x0 = (int)floor(cx) - w / 2, y0 = (int)floor(cy) - hh / 2;
        if (x0 < 0) x0 = 0;
        if (x0 > nx - 1 - w) x0 = nx - 1 - w;
        if (y0 < 0) y0 = 0;
        if (y0 > ny - 1 - hh) y0 = ny - 1 - hh;
        /* pins, merged per G-cell (union of pin spans) */
        scratch_reserve(&s, k);
        int m = 0;
        for (int i = 0; i < k; i++) {
            int px = x0 + (int)rng_int(&rng, 0, w), py = y0 + (int)rng_int(&rng, 0, hh);
            int lay = rng_u01(&rng) < 0.9 ? 0 : 1;
            int j;
            for (j = 0; j < m; j++) if (s.nodes[j].x == px && s.nodes[j].y == py) break;
            if (j < m) {
                if (lay < s.nodes[j].lo) s.nodes[j].lo = lay;
                if (lay > s.nodes[j].hi) s.nodes[j].hi = lay;
            } else {
                s.nodes[m].x = px; s.nodes[m].y = py; s.nodes[m].lo = lay; s.nodes[m].hi = lay; m++;
            }
        }
        /* Prim MST from node 0; Manhattan distance; ties to the lower index */
        for (int i = 0; i < m; i++) { s.in[i] = 0; s.dist[i] = 0x7fffffff; s.par[i] = -1; }
        s.dist[0] = 0;
        int cnt = 0;
        for (int it = 0; it < m; it++) {
            int best = -1;
            for (int i = 0; i < m; i++)
                if (!s.in[i] && (best < 0 || s.dist[i] < s.dist[best])) best = i;
            s.in[best] = 1; s.order[cnt++] = best;
            for (int i = 0; i < m; i++) {
                if (s.in[i]) continue;
                int d = iabs(s.nodes[i].x - s.nodes[best].x) + iabs(s.nodes[i].y - s.nodes[best].y);
                if (d < s.dist[i]) { s.dist[i] = d; s.par[i] = best; }
            }
        }
        /* one pass of 3-terminal median Steiner insertion over the original nodes */
        int morig = m;
        if (p->steiner) {
            for (int ui = 0; ui < morig; ui++) {
                int u2 = s.order[ui];
                int c1 = -1, c2 = -1;
                for (int i = 0; i < m; i++)
                    if (s.par[i] == u2) { if (c1 < 0) c1 = i; else if (c2 < 0) c2 = i; }
                if (c2 < 0) continue;
                int sx = med3(s.nodes[u2].x, s.nodes[c1].x, s.nodes[c2].x);
                int sy = med3(s.nodes[u2].y, s.nodes[c1].y, s.nodes[c2].y);
                if (has_node_at(s.nodes, m, sx, sy)) continue;
                s.nodes[m].x = sx; s.nodes[m].y = sy; s.nodes[m].lo = -1; s.nodes[m].hi = -1;
                s.par[m] = u2; s.par[c1] = m; s.par[c2] = m;
                m++;
            }
        }
        /* DFS preorder renumbering from root 0, children in index order */
        int sp = 0, nid = 0;
        s.stack[sp++] = 0;
        while (sp > 0) {
            int v = s.stack[--sp];
            s.newidx[v] = nid++;
            /* push children in reverse index order so lower index is visited first */
            for (int i = m - 1; i >= 0; i--) if (s.par[i] == v) s.stack[sp++] = i;
        }
        push_reserve(out, M + m);
        for (int i = 0; i < m; i++) {
            int ni = (int)M + s.newidx[i];
            out->x[ni] = (int16_t)s.nodes[i].x;
            out->y[ni] = (int16_t)s.nodes[i].y;
            if (literal) { out->pin_lo[ni] = -1; out->pin_hi[ni] = -1; }
            else { out->pin_lo[ni] = (int8_t)s.nodes[i].lo; out->pin_hi[ni] = (int8_t)s.nodes[i].hi; }
            out->parent[ni] = s.par[i] < 0 ? -1 : s.newidx[s.par[i]];
        }
        M += m;
        out->node_offset[n + 1] = (int32_t)M;
    }
    out->num_nodes = (int32_t)M;
    free(s.nodes); free(s.par); free(s.newidx); free(s.order); free(s.stack); free(s.dist); free(s.in);
    return 0;
}

void fgr_gen_free(gen_design* d) {
    free(d->edge_capacity); free(d->node_offset); free(d->x); free(d->y);
    free(d->pin_lo); free(d->pin_hi); free(d->parent);
    memset(d, 0, sizeof(*d));
}
