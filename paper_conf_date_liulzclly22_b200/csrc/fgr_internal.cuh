// fgr_internal.cuh — internal state and device helpers of libfastgr (not part of the ABI).
//
// HBM layout.  For each direction d in {H, V} the wire edges of
// the d-layers are stored "sector-major": one line (a row for H, a column for
// V) is a run of `len` positions, each position holding W_d words, one per
// d-layer slot (W_d = number of d-layers rounded up to a power of two >= 4):
//     H:  element (y, x, slot) at ((y*nx + x)*WH + slot)   edge (x,y)-(x+1,y)
//     V:  element (x, y, slot) at ((x*ny + y)*WV + slot)   edge (x,y)-(x,y+1)
// so all H layers of one G-cell edge sit in one 32-byte sector (L = 9: 5 H
// layers -> WH = 8) and a tree-DP gather of a prefix position is one sector.
// Arrays per direction: D (int32 demand), C (uint8 capacity), P (uint32
// segment-local exclusive prefix of the edge cost), ST (uint32 per-segment
// totals), SB (uint32 exclusive prefix of segment totals).  A segment is 32
// consecutive positions of one line; the global prefix of position p is
// SB[seg(p)] + P[p], so a leg cost is a difference of two such sums (exact in
// uint32 modular arithmetic because every true prefix is < 2^32, R19).
#pragma once

#include <cuda_runtime.h>
#include <nccl.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "fastgr.h"

#define FGR_SEG 32          // positions per scan segment (one warp)
#define FGR_SEG_SHIFT 5
#define FGR_CHUNK_SEGS 8    // segments per refresh task (one warp)
#define FGR_INF 0x7FFFFFFFu // "impossible" cost; finite costs are < FGR_INF (R19)
#define FGR_MAXL 16
#define FGR_SMALL_NET 32    // nets with <= this many nodes take the lane-group path
#define FGR_MID_NET 8       // ... with a node capacity of 8 (3..8 nodes) or 32 (9..32 nodes)
#define FGR_SIDE_STREAMS 7
#define FGR_CTA_THREADS 256
#define FGR_WARPS_PER_CTA (FGR_CTA_THREADS / 32)

// ------------------------------------------------------------------ device views
struct DirView {            // one direction's arrays
    int32_t* D;
    const uint8_t* C;
    uint32_t* P;
    uint32_t* ST;
    uint32_t* SB;
    int len;                // positions per line (nx for H, ny for V)
    int lines;              // ny for H, nx for V
    int W;                  // words per position
    int cnt;                // layers of this direction
    int nseg;               // segments per line
    int seg_base;           // global segment index of this direction's first segment
    int line_base;          // index of this direction's first line in the line counters
};

struct GridView {
    DirView h, v;
    int nx, ny, L, S, len_cost;
    const int32_t* table;   // [L][2S+1]
    uint8_t* dseg;          // [total segments] dirty flag (plain stores by the commit)
    uint8_t* dline;         // [ny + nx] the line has a dirty segment
    uint32_t* linedone;     // [ny + nx] chunks of the line refreshed in this launch
    unsigned long long* stats;  // [4] device counters (refresh segments, ...)
    uint8_t dir[FGR_MAXL];
    uint8_t slot[FGR_MAXL]; // index of layer l among the layers of its direction
    uint8_t layer_of_slot[2][FGR_MAXL];
    uint32_t viapre[FGR_MAXL + 1];  // V(lo,hi) = viapre[hi] - viapre[lo]
};

struct NetsView {
    const int32_t* off;
    const int16_t* x;
    const int16_t* y;
    const int8_t* plo;
    const int8_t* phi;
    const int32_t* par;
};

// ------------------------------------------------------------------ host state
// Heavy-path decomposition of every net routed by k_dp_hld (dp_hld.cu), computed once per
// stage by k_hld_prep.  Global arrays indexed by global node index (a0 + local), values
// net-local (uint16): heavy child (0xFFFF = leaf), child CSR (cs[a0+v] .. cs[a0+v+1], with
// cs of local m implied = m - 1), path nodes pn (paths stored bottom -> head, paths ordered
// by light depth, deepest first), path starts po[a0 + q] (q < npaths; the end of the last is m),
// path light depth pr[a0 + q]; info[net] = npaths | rounds << 16.
struct HldPrep {
    const uint16_t* hv;
    const uint16_t* cs;
    const uint16_t* cl;
    const uint16_t* pn;
    const uint16_t* po;
    const uint8_t* pr;
    const int32_t* info;
    const uint8_t* ld;     // light depth of every node (= the round of its path)
    const uint16_t* lf;    // leaves (path bottoms) by descending depth, ties by index (k_dp_tree), [a0 + q], q < npaths
};

// Per-node results of the large-net tree analysis (global, indexed by global node index).
struct Prep {
    const uint16_t* cs;    // child CSR start (net-local); cs of local m is m - 1 and not stored
    const uint16_t* cl;    // child list
    const uint16_t* hv;    // heavy child
    const uint16_t* bot;   // bottom of the path topped by the node
    const uint16_t* pq;    // path queue (path tops, deepest first)
    const int32_t* npaths; // [num_nets]
    const uint16_t* rpos;  // index along the root path (0xFFFF off it)
    HldPrep hld;           // heavy-path decomposition for k_dp_hld (the default large-net kernel)
};

// Hybrid L+Z tables of the current route call (hybrid.cu).  Slots number the hybrid
// edges; M[s][lt][ls] is the edge's transfer cost from layer ls at the child to lt at
// the parent (legs + bend vias, FGR_INF if no candidate), A[s][lt][ls] its Z argmin
// (mid | lb << 16) or 0xFFFFFFFF for the L shape.
struct HybView {
    const int32_t* net;    // [num_nets] first slot of the net, -1 = no hybrid edge (NULL = L only)
    const int32_t* slot;   // [num_nodes] slot of the node's edge, -1 = L edge (valid in nets with net >= 0)
    const uint32_t* M;
    const uint32_t* A;
};

struct HybState {
    bool active = false;
    int nslots = 0;
    int32_t* net = nullptr;
    int32_t* slot = nullptr;
    int32_t* list = nullptr;   // [nslots] global child node of the edge
    int32_t* par = nullptr;    // [nslots] global parent node
    uint32_t* M = nullptr;
    uint32_t* A = nullptr;
    std::vector<int> boff;     // host: slot offsets per batch
    bool cached = false;       // tables valid for (key_exec, key_t1, key_t2) of fgr_route_all
    const int32_t* key_exec = nullptr;
    int key_t1 = 0, key_t2 = 0;
    HybView view() const {
        HybView v;
        v.net = active ? net : nullptr; v.slot = slot; v.M = M; v.A = A;
        return v;
    }
};

struct PlanCache {
    bool valid = false;
    fgr_nets nets{};
    const int32_t* order = nullptr;
    const int32_t* batch_offset = nullptr;
    int num_batches = 0;
    // host mirrors, per batch
    int* h_off = nullptr;      // [B+1]
    int* h_nlarge = nullptr;   // [B]
    int* h_maxm = nullptr;     // [B] max nodes of a large net in the batch
    int* h_ntwo = nullptr;     // [B] 2-node nets (the tail of each batch in exec order)
    int* h_n9 = nullptr;       // [B] nets with 9..32 nodes
    int* h_lsplit = nullptr;   // [B][5] large nets with more than fgr_large_limit, 512, 256, 128, 64 nodes
    const int32_t* exec = nullptr;  // exec order actually used (order itself, or a re-sorted copy)
    bool prep_valid = false;        // large-net tree analysis computed for these nets
    Prep prep{};
    long long* h_segb = nullptr;  // [B] upper bound on segments the batch can dirty
    int cap = 0;
};

extern unsigned long long g_scratch_gen;   // bumped whenever a scratch buffer is (re)allocated

// Captured single-GPU batch loop of fgr_route_all (route.cu): valid while every input of
// the loop's launches is unchanged (key, host batch mirrors, scratch generation).
struct RouteGraph {
    bool use = true;
    cudaGraphExec_t exec = nullptr;
    cudaStream_t cap = nullptr;       // private stream the loop is captured on
    std::vector<long long> key;       // pointers, sizes, policy, pattern, initial full-dirty flag, scratch gen
    std::vector<long long> mirror;    // h_off, h_nlarge, h_maxm, h_ntwo, h_n9, h_lsplit, h_segb
    long long launches = 0;           // library kernel launches in the captured loop
    std::vector<long long> seen_key, seen_mirror;   // the previous direct run (capture on the next equal call)
};

struct Scratch {            // grow-only device scratch
    void* p = nullptr;
    size_t bytes = 0;
};

#include <vector>

struct Profiler {
    bool on = false;
    std::vector<cudaEvent_t> pool;        // start/stop pairs
    std::vector<int> cls;                 // class of each recorded pair
    size_t used = 0;
    double ms[FGR_PROF_CLASSES] = {0};
    long long launches[FGR_PROF_CLASSES] = {0};
};

struct fgr_grid {
    int device = 0;
    int nx = 0, ny = 0, L = 0, S = 0, len_cost = 0;
    uint8_t dir[FGR_MAXL];
    int32_t layer_capacity[FGR_MAXL];
    int32_t via_cost[FGR_MAXL];
    int32_t ovf_weight[FGR_MAXL];
    double slope = 1.0;
    int nH = 0, nV = 0, WH = 0, WV = 0;
    GridView view{};
    // device allocations
    void* mem = nullptr;        // one slab for the grid arrays
    size_t mem_bytes = 0;
    int32_t* d_table = nullptr;
    unsigned long long* d_stats = nullptr;
    bool full_dirty = true;     // next refresh must rescan everything
    bool broken = false;
    int total_segs = 0;
    // plan scratch
    Scratch s_plan[14];
    PlanCache cache;
    // multi-GPU
    ncclComm_t comm = nullptr;
    int rank = 0, world = 1;
    Scratch s_rec[4];
    Scratch s_prep;
    Scratch s_hldp;             // k_hld_prep outputs (per stage)
    Scratch s_hldt;             // k_hld_prep temporaries for nets too large for shared memory
    Scratch s_hldw;             // per large-net unit: k_dp_hld workspaces (per CTA), k_tree_legs leg rows
    fgr_stats stats{};
    int max_smem = 0;
    int num_sms = 0;
    Profiler prof;
    // size classes of one batch run side by side: 3 small-net classes + 4 more large-net size buckets
    cudaStream_t side[FGR_SIDE_STREAMS] = {};
    cudaEvent_t ev_fork = nullptr, ev_join[FGR_SIDE_STREAMS] = {};
    // hybrid L+Z pattern routing (fgr_set_pattern): edges with t1 <= HPWL <= t2; t1 > t2 = L only
    int hyb_t1 = 1, hyb_t2 = 0;
    // large-net DP kernel selection (fgr_set_dp_policy)
    int dp_policy = FGR_DP_AUTO;
    int flow_max = 64;
    // multi-GPU exchange (fgr_set_exchange): batches below split_min nets are routed whole on every
    // rank; emu_world > 1 runs the exchange path with that many emulated ranks on one device
    int split_min = 2048;
    int emu_world = 0;
    HybState hy;
    RouteGraph rg;
    Scratch s_hyb[3];
    Scratch s_rip[6];          // rip-up extraction and task graph (ripup.cu)
};

// Profiling brackets around a launch (no-ops unless fgr_profile_enable(grid, 1)).
int fgr_prof_begin(fgr_grid* g, int cls, cudaStream_t st);
void fgr_prof_end(fgr_grid* g, int slot, cudaStream_t st);
enum { PROF_REFRESH = 0, PROF_DP_SMALL, PROF_DP_LARGE, PROF_COMMIT, PROF_PRE, PROF_SORT, PROF_COLOR, PROF_PLAN_OTHER,
       PROF_EXCHANGE, PROF_HYBRID };

// ------------------------------------------------------------------ host helpers
fgr_status fgr_set_error(fgr_status s, const char* fmt, ...);
// host mirrors of the plan's per-batch sizes, pinned (async D2H copies); capacity >= B + 1 batches
cudaError_t fgr_mirrors_reserve(PlanCache& c, int B);
void fgr_mirrors_free(PlanCache& c);
fgr_status fgr_cuda_fail(fgr_grid* g, cudaError_t e, const char* where);
void* fgr_scratch(Scratch& s, size_t bytes, cudaError_t* err);

#define FGR_CHECK_CUDA(g, expr)                                        \
    do {                                                               \
        cudaError_t _e = (expr);                                       \
        if (_e != cudaSuccess) return fgr_cuda_fail((g), _e, #expr);   \
    } while (0)

// launchers (defined in the .cu files)
cudaError_t fgr_launch_refresh(fgr_grid* g, cudaStream_t st, bool full);
cudaError_t fgr_launch_refresh_sized(fgr_grid* g, cudaStream_t st, bool full, long long max_tasks);
// list = [large (> 32 nodes) | midL (9..32) | midS (3..8) | two (2 nodes)] nets, contiguous
cudaError_t fgr_launch_dp(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int nlarge,
                          int nmidL, int nmidS, int ntwo, int maxm_large, uint32_t* seg_out, uint32_t* cost_out,
                          uint32_t* rec_seg, const int32_t* rec_off, uint32_t* rec_cost, int list_base,
                          bool commit, const Prep* prep, const int* lsplit = nullptr);
cudaError_t fgr_launch_large_prep(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int count,
                                  int maxm, uint16_t* cs, uint16_t* cl, uint16_t* hv, uint16_t* bot, uint16_t* pq,
                                  uint16_t* rpos, int32_t* np);
cudaError_t fgr_launch_commit(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int count,
                              const uint32_t* rec_seg, const int32_t* rec_off, int list_base);
fgr_status fgr_hyb_prepare(fgr_grid* g, cudaStream_t st, const NetsView& nv, int num_nets, int num_nodes,
                           const int32_t* exec, int R, const int32_t* boff, int nb, int32_t* zmid);
cudaError_t fgr_launch_hyb_tm(fgr_grid* g, cudaStream_t st, const NetsView& nv, int slot0, int n);
cudaError_t fgr_launch_hyb_zmid(fgr_grid* g, cudaStream_t st, const uint32_t* seg, int32_t* zmid);
size_t fgr_dp_smem_large(const fgr_grid* g, int m);
struct Out;
cudaError_t fgr_launch_walk(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int mc,
                            const Out& o, bool commit);
cudaError_t fgr_launch_flow(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                            const Out& o, bool commit, const Prep& prep);
int fgr_flow_max_nodes(const fgr_grid* g);
int fgr_large_limit(const fgr_grid* g);
int fgr_top_limit(const fgr_grid* g);   // size above which nets take k_dp_hld (policy dependent)
cudaError_t fgr_launch_hld_prep(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int count,
                                int maxm, uint16_t* hv, uint16_t* cs, uint16_t* cl, uint16_t* pn, uint16_t* po,
                                uint8_t* pr, int32_t* info, uint8_t* ld, uint16_t* lf);
// k_dp_tree (dp_tree.cu): nets of FGR_SMALL_NET+1 .. fgr_tree_cap(g) nodes; commit = launch k_commit_nets after it
// legs: NULL (the kernel gathers its legs) or the rows of fgr_launch_tree_legs (net i at legs + i * 2 * legs_maxm * L)
cudaError_t fgr_launch_tree(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                            const Out& o, bool commit, const HldPrep& hp, const uint32_t* legs, int legs_maxm);
// k_tree_legs: leg rows of n nets (<= maxm nodes) into legs [n][2][maxm][L], one task per thread on many SMs
cudaError_t fgr_launch_tree_legs(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                                 uint32_t* legs);
// S6 for nets routed without an in-kernel commit: one thread per tree edge (reads seg or the route records)
cudaError_t fgr_launch_commit_nets(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                                   const Out& o);
int fgr_tree_cap(const fgr_grid* g);
// ws: global workspace of fgr_hld_ws_bytes(g, n, maxm) bytes (distinct per concurrent launch)
cudaError_t fgr_launch_hld(fgr_grid* g, cudaStream_t st, const NetsView& nv, const int32_t* list, int n, int maxm,
                           const Out& o, bool commit, const HldPrep& hp, unsigned char* ws);
size_t fgr_hld_ws_bytes(const fgr_grid* g, int n, int maxm);

// Output of a DP launch: direct (by node / net id) or route records (multi-GPU).
struct Out {
    uint32_t* seg;        // [num_nodes] by global node index (direct mode)
    uint32_t* cost;       // [num_nets] by net id (direct mode)
    uint32_t* rec_seg;    // record mode: rec_seg[rec_off[list_base + idx] + local]
    const int32_t* rec_off;
    uint32_t* rec_cost;   // record mode: rec_cost[list_base + idx]
    int list_base;
};

static inline NetsView fgr_nets_view(const fgr_nets* n) {
    NetsView v;
    v.off = n->node_offset; v.x = n->x; v.y = n->y; v.plo = n->pin_lo; v.phi = n->pin_hi; v.par = n->parent;
    return v;
}

// ------------------------------------------------------------------ device helpers
// min(a + b, INF) for a, b <= INF: one DPX VIADDMNMX on sm_100a.
__device__ __forceinline__ uint32_t sat_add(uint32_t a, uint32_t b) { return __viaddmin_u32(a, b, FGR_INF); }

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }

// Programmatic dependent launch (sm_90+): let the next kernel on the stream start its
// demand-independent prologue early; wait for the previous kernel before touching its
// results.  Both are no-ops when the launch did not request PDL.
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

template <int N>
struct U32Vec { uint32_t v[N]; };
