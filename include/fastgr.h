/*
 * fastgr.h — C ABI of the B200-native batched 3-D L-shape pattern router
 * (FastGR pattern-routing stage: PAPER.md §III-C/§III-D).
 *
 * Plain C: pointers and sizes only, no exceptions and no torch types cross this
 * boundary.  Every entry point returns an fgr_status; on non-OK, fgr_last_error()
 * returns a thread-local message.  A non-OK status from validation leaves the
 * grid's demand untouched.  A CUDA or NCCL failure moves the handle to
 * FGR_ERR_STATE (every later call on it returns FGR_ERR_STATE).
 *
 * Streams: every call enqueues on the caller's stream (cudaStream_t passed as
 * void*, e.g. torch.cuda.current_stream().cuda_stream; NULL = legacy default).
 * Only fgr_plan, fgr_route_batch and fgr_run_host synchronise that stream
 * (plan returns num_batches to the host; route_batch sizes its launch).
 *
 * Problem statement (§II-A): a grid graph of G-cells with L
 * metal layers, each with one preferred direction (L203-206); wire edges join
 * adjacent G-cells on one layer and carry capacity (tracks) and demand; via
 * edges join layers at one G-cell.  A multipin net is a set of pin points on
 * the grid (L226-227) given as a tree of two-pin nets (L227-233).
 */
#ifndef FASTGR_H
#define FASTGR_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define FGR_API __attribute__((visibility("default")))
#else
#define FGR_API
#endif

typedef enum {
    FGR_OK = 0,
    FGR_ERR_INVALID = 1,   /* malformed input (see each call)                           */
    FGR_ERR_RANGE = 2,     /* a cost could overflow the integer ranges (R19)   */
    FGR_ERR_OOM = 3,       /* device allocation failed                                   */
    FGR_ERR_CUDA = 4,      /* CUDA runtime error                                         */
    FGR_ERR_NCCL = 5,      /* NCCL error                                                 */
    FGR_ERR_STATE = 6      /* handle unusable after an earlier CUDA/NCCL failure, or a
                              call made in the wrong state (e.g. comm not initialised)   */
} fgr_status;

/* Message for the last non-OK status returned on this thread ("" if none). */
FGR_API const char* fgr_last_error(void);
FGR_API const char* fgr_version(void);

typedef struct fgr_grid fgr_grid;

/*
 * Grid description (cost scheme L556-563 = DESIGN.md
 * readings R1/R2).  All integer costs:
 *   edge cost   ec_l(e) = len_cost + T_l[clamp(cap_l(e) - dem_l(e), -S, S)]
 *   T_l[s]      = round_half_away(ovf_weight[l] / (1 + exp(logistic_slope * s)))
 *   via stack   V(lo,hi) = sum_{k=lo}^{hi-1} via_cost[k]
 * Host pointers are read during fgr_grid_create only.
 */
typedef struct {
    int32_t nx, ny, nlayers;           /* G-cell dims 2..32767; 2 <= nlayers <= 16            */
    const uint8_t* dir;                /* host [nlayers]: 0 = horizontal, 1 = vertical; needs
                                          at least one H and one V layer                       */
    const int32_t* layer_capacity;     /* host [nlayers]: tracks per wire edge, 0..255         */
    const uint8_t* edge_capacity;      /* DEVICE [nlayers][ny][nx] per-edge override or NULL;
                                          copied at create.  Entry (l,y,x) is edge (x,y)-(x+1,y)
                                          on an H layer, (x,y)-(x,y+1) on a V layer.           */
    int32_t len_cost;                  /* per unit wire edge, >= 0 (default 64)                */
    const int32_t* via_cost;           /* host [nlayers-1], >= 0 (default 32)                  */
    const int32_t* ovf_weight;         /* host [nlayers], >= 0 (default 4096)                  */
    double logistic_slope;             /* per track of slack (default 1.0)                     */
    int32_t slack_clamp;               /* S, 0..1024 (default 64)                              */
} fgr_grid_desc;

/* Host-only: the integer logistic table T as the library builds it,
 * table[l*(2S+1) + (s+S)] for s in [-S,S].  Needs no GPU. */
FGR_API fgr_status fgr_cost_table(const fgr_grid_desc* desc, int64_t* table);

/* Allocates the grid on `device` (demand = 0).  Errors: INVALID (desc), RANGE
 * ((len_cost + max W) * max(nx,ny) >= 2^31 - 1, or the via costs sum to >= 2^24),
 * OOM, CUDA.  Caller owns *out. */
FGR_API fgr_status fgr_grid_create(const fgr_grid_desc* desc, int device, void* stream, fgr_grid** out);
FGR_API fgr_status fgr_grid_destroy(fgr_grid* grid);

/* Demand in the dense layout int32 [nlayers][ny][nx] (same entry convention as
 * edge_capacity; unused entries (x = nx-1 on H, y = ny-1 on V) are ignored on set
 * and returned as 0).  DEVICE pointers.  set(NULL) zeroes the demand.  Setting the
 * demand marks every cost stale (the next route does a full refresh). */
FGR_API fgr_status fgr_grid_set_demand(fgr_grid* grid, const int32_t* demand, void* stream);
FGR_API fgr_status fgr_grid_get_demand(fgr_grid* grid, int32_t* demand, void* stream);

/*
 * Nets: DEVICE pointers owned by the caller, valid for the duration of the call.
 * CSR over nets: net i has nodes node_offset[i] .. node_offset[i+1]-1 (>= 1 node).
 * Local node 0 is the root; parent[] is net-local with parent[j] in [0, j-1] for
 * j >= 1 (so any descending index order is children-first) and -1 at j = 0.
 * x,y are G-cell coordinates; [pin_lo, pin_hi] is the node's pin layer span
 * (-1,-1 = Steiner node, or paper-literal 2-D pin).  A node and its parent must
 * lie in different G-cells (merge coincident nodes, union their spans).
 * Single-node nets are trivial: never batched, no demand, cost 0.
 */
typedef struct {
    int32_t num_nets, num_nodes;
    const int32_t* node_offset;        /* [num_nets+1], node_offset[0] = 0                     */
    const int16_t* x;                  /* [num_nodes]                                           */
    const int16_t* y;                  /* [num_nodes]                                           */
    const int8_t* pin_lo;              /* [num_nodes]                                           */
    const int8_t* pin_hi;              /* [num_nodes]                                           */
    const int32_t* parent;             /* [num_nodes]                                           */
} fgr_nets;

/*
 * fgr_plan — conflict-free batching (Algorithm 1, §III-C
 * L468-504): non-trivial nets sorted by ascending bounding-box half-perimeter
 * (over all tree nodes), ties by net id (L1305-1308; R12); a net
 * joins the first batch holding no net whose closed bounding box touches its
 * own (R13).  Computed on the device as first-fit colouring, identical to the
 * literal repeated passes of Algorithm 1 (proof).
 *   batch_of_net [num_nets]   DEVICE out: batch id, -1 for trivial nets
 *   order        [num_nets]   DEVICE out: net ids grouped by batch (batch 0 first);
 *                             trivial nets last; order inside a batch is unspecified
 *   batch_offset [num_nets+1] DEVICE out: batch b = order[batch_offset[b] .. batch_offset[b+1])
 *   num_batches               HOST out
 * Errors: INVALID (malformed nets: the message names the first bad net), RANGE
 * (a net's worst-case cost could reach 2^31, or a net of more than 65535 nodes),
 * OOM, CUDA.  Synchronises `stream`.  The plan (host batch sizes, the tree
 * decompositions of the large nets, the hybrid tables, a captured batch-loop
 * graph) is cached by the identity of the nets and output buffers: after
 * rewriting the nets' arrays in place, call fgr_plan again before routing.
 */
FGR_API fgr_status fgr_plan(fgr_grid* grid, const fgr_nets* nets, int32_t* batch_of_net, int32_t* order,
                            int32_t* batch_offset, int32_t* num_batches, void* stream);

/*
 * fgr_route_batch — route one conflict-free batch on the current demand:
 * cost refresh of stale rows/columns, the per-net tree DP (Eqs. (1)-(7),
 * PAPER.md L582-756), backtrack, and the +1 demand commit of every chosen leg.
 *   net_ids [count] DEVICE: nets of the batch (their bounding boxes must be
 *                   pairwise disjoint — not checked; overlapping boxes give a
 *                   result that depends on scheduling)
 *   seg_out [num_nodes] DEVICE out: for each non-root node v (edge v -> parent u):
 *           bend | ls<<8 | lt<<16 | straight<<24.  bend 0: bend point (x_u, y_v),
 *           leg 1 horizontal on layer ls, leg 2 vertical on lt; bend 1: bend point
 *           (x_v, y_u), leg 1 vertical on ls, leg 2 horizontal on lt; straight:
 *           one leg on ls = lt.  Roots get 0xFFFFFFFF.  Other nodes untouched.
 *   net_cost [num_nets] DEVICE out: routed cost of each listed net.
 * Synchronises `stream` once (launch sizing).  Ignores any communicator.
 */
FGR_API fgr_status fgr_route_batch(fgr_grid* grid, const fgr_nets* nets, const int32_t* net_ids, int32_t count,
                                   uint32_t* seg_out, uint32_t* net_cost, void* stream);

/*
 * fgr_set_pattern — candidate pattern set of later fgr_route_* / fgr_run_host_ex
 * calls on this grid.  A bent tree edge v -> u whose two-pin half perimeter
 * |x_v - x_u| + |y_v - y_u| lies in [hybrid_t1, hybrid_t2] takes the HYBRID
 * L+Z patterns (§III-E/F, L758-1092: the two L shapes plus every Z
 * shape whose two bend points lie strictly inside the edge's box; Eq. (8) path
 * cost, Eqs. (9)-(14) candidate flows, Eq. (10) merge); every other edge takes
 * the L patterns.  This is the paper's selection technique (§IV-D;
 * FastGRH uses t1 = 100, t2 = 500).  hybrid_t1 > hybrid_t2 (the default,
 * 1 > 0) = L patterns only (FastGRL).  A chosen Z is reported as seg bend 2
 * (HVH: leg 1 horizontal on ls along row y_v to x = mid, leg 2 vertical on lb
 * along column mid, leg 3 horizontal on lt along row y_u) or bend 3 (VHV: leg 1
 * vertical on ls along column x_v to y = mid, leg 2 horizontal on lb along row
 * mid, leg 3 vertical on lt along column x_u), with mid | lb << 16 in zmid_out.
 * Tie order of equal costs: smallest ls, then the L shape, then Z by increasing
 * mid, then smallest lb (R25).  Errors: INVALID (window outside
 * [0, 65534] when enabled).  Host-only; takes effect at the next route call.
 */
FGR_API fgr_status fgr_set_pattern(fgr_grid* grid, int32_t hybrid_t1, int32_t hybrid_t2);

/*
 * fgr_set_dp_policy — which tree-DP kernel routes nets of more than 32 nodes
 * (all kernels compute the same DP, §III-D Eqs. (1)-(7), and give
 * bit-identical routes; the choice only changes speed):
 *   FGR_DP_AUTO  (default) the leaf-to-root dataflow kernel k_dp_tree while the
 *                net's tables fit one SM's shared memory (~1.1k nodes at L = 9),
 *                above that the heavy-path contraction kernel k_dp_hld (global
 *                workspace, any size up to 65535 nodes);
 *   FGR_DP_HEAVY the previous kernels: nets of up to flow_max nodes the tree-
 *                dataflow kernel k_dp_flow, bigger nets the heavy-path kernel
 *                k_dp_large (~1.3k nodes at L = 9), above that k_dp_hld;
 *   FGR_DP_HLD   k_dp_hld for every net of > 32 nodes.
 * flow_max in [33, 65535] (default 64; used by FGR_DP_HEAVY).  Errors: INVALID.
 * Host-only; takes effect at the next route call.
 */
#define FGR_DP_AUTO 0
#define FGR_DP_HEAVY 1
#define FGR_DP_HLD 2
FGR_API fgr_status fgr_set_dp_policy(fgr_grid* grid, int32_t policy, int32_t flow_max);

/* fgr_route_batch with the Z middles: zmid_out [num_nodes] DEVICE out (may be NULL):
 * for the listed nets' nodes, mid | lb << 16 of an edge routed as a Z shape
 * (seg bend 2 or 3), -1 otherwise.  Same synchronisation and errors. */
FGR_API fgr_status fgr_route_batch_ex(fgr_grid* grid, const fgr_nets* nets, const int32_t* net_ids, int32_t count,
                                      uint32_t* seg_out, int32_t* zmid_out, uint32_t* net_cost, void* stream);

/*
 * fgr_route_all — the pattern-routing stage: batches in sequence (PAPER.md
 * L504-512, Fig. 7), each routed on the demand left by all earlier batches.
 * order/batch_offset/num_batches as returned by fgr_plan for the same nets.
 * seg_out [num_nodes] and net_cost [num_nets] are fully written (trivial nets:
 * seg 0xFFFFFFFF, cost 0).  With a communicator (fgr_comm_init, world > 1),
 * each batch of at least split_min nets is split across ranks by tree edges
 * (fgr_split_batch) and the routes are exchanged with one NCCL all-reduce per
 * batch; smaller batches are routed whole on every rank (fgr_set_exchange).  Every
 * rank ends with identical outputs and demand, bitwise equal to world = 1.  (A
 * communicator of world 1 takes the same exchange path; fgr_set_exchange's
 * emulate_world runs it with k emulated ranks on one GPU.)  The exchange path
 * synchronises the stream once per call (record offsets and the edge split);
 * without it there is no host synchronisation when the arguments are those of
 * the grid's last fgr_plan call.  The plan cache is keyed on the identity of the
 * `nets` device pointers and order/batch_offset: after rewriting those buffers in
 * place, call fgr_plan again.
 */
FGR_API fgr_status fgr_route_all(fgr_grid* grid, const fgr_nets* nets, const int32_t* order,
                                 const int32_t* batch_offset, int32_t num_batches, uint32_t* seg_out,
                                 uint32_t* net_cost, void* stream);

/* fgr_route_all with the Z middles: zmid_out [num_nodes] DEVICE out (may be NULL),
 * fully written: mid | lb << 16 for edges routed as a Z shape, -1 elsewhere.
 * With hybrid patterns on, one host synchronisation per new (plan, window). */
FGR_API fgr_status fgr_route_all_ex(fgr_grid* grid, const fgr_nets* nets, const int32_t* order,
                                    const int32_t* batch_offset, int32_t num_batches, uint32_t* seg_out,
                                    int32_t* zmid_out, uint32_t* net_cost, void* stream);

/*
 * fgr_split_batch — the multi-GPU split rule fgr_route_all applies to one batch
 * (host-only, no GPU).  The batch's `count` nets are in exec
 * order, large nets first (`nlarge` of them).  edge_prefix [count+1] HOST in (may
 * be NULL): edge_prefix[i] = tree edges of the batch's first i nets.  Rank r of
 * `world` routes the large nets [out[0], out[1]) and the small nets [out[2],
 * out[3]) (indices into the batch): contiguous, disjoint and covering, balanced by
 * tree edges (by net count when edge_prefix is NULL).  A batch of fewer than
 * split_min nets is not split: out = {0, nlarge, nlarge, count} on every rank and
 * out[4] = 1 (every rank routes it whole and no exchange is needed); else out[4] = 0.
 * out5 [5] HOST out.  Errors: INVALID.
 */
FGR_API fgr_status fgr_split_batch(int32_t count, int32_t nlarge, const int64_t* edge_prefix, int32_t split_min,
                                   int32_t rank, int32_t world, int32_t* out5);

/*
 * fgr_set_exchange — multi-GPU exchange settings of later fgr_route_all(_ex) calls.
 *   split_min (default 2048): batches of fewer nets are routed whole on every
 *       rank instead of split + all-reduced (a batch's latency is its biggest
 *       net; a collective per small batch only adds latency).  0 = split every batch.
 *   emulate_world: 0 or 1 = off; k > 1 = TEST MODE on a grid without a
 *       communicator: fgr_route_all takes the exchange path with k emulated ranks on
 *       this device (every rank's chunk routed into the shared route records, which
 *       then hold what the NCCL SUM all-reduce would; then the commit from the
 *       records), so the split, record and commit code runs on one GPU.
 * Host-only; takes effect at the next route call.  Errors: INVALID.
 */
FGR_API fgr_status fgr_set_exchange(fgr_grid* grid, int32_t split_min, int32_t emulate_world);

/*
 * fgr_set_graph — replay the single-GPU batch loop of fgr_route_all(_ex) as a CUDA
 * Graph (on = 1, the default) or issue it launch by launch (on = 0).  The batches
 * run in sequence either way (one kernel invocation per batch);
 * the graph only removes the host issue cost and the inter-launch gaps.  A call
 * whose plan (host batch sizes), nets/output pointers, stream, DP policy and
 * pattern equal those of the previous call is captured once and then replayed;
 * any change re-runs the loop directly.  Not used with a communicator, with
 * emulated ranks or while the profiler is on.  Routes are identical in both modes.
 * Errors: INVALID (NULL grid).  Host-only.
 */
FGR_API fgr_status fgr_set_graph(fgr_grid* grid, int32_t on);

/* Multi-GPU (one process per GPU).  fgr_comm_unique_id fills 128 bytes on the
 * root rank; broadcast them (e.g. torch.distributed) and call fgr_comm_init on
 * every rank with the grid already created on that rank's device. */
FGR_API fgr_status fgr_comm_unique_id(void* out128);
FGR_API fgr_status fgr_comm_init(fgr_grid* grid, const void* nccl_unique_id, int rank, int world);

/*
 * fgr_run_host — end-to-end convenience over HOST buffers: copies the nets to
 * the device, resets the demand to zero, plans, routes all batches, and copies
 * the per-node segments and per-net costs back.  Host arrays as in fgr_nets;
 * seg_out [num_nodes], net_cost [num_nets], num_batches may be NULL.
 * Synchronises `stream`.
 */
FGR_API fgr_status fgr_run_host(fgr_grid* grid, int32_t num_nets, int32_t num_nodes, const int32_t* node_offset,
                                const int16_t* x, const int16_t* y, const int8_t* pin_lo, const int8_t* pin_hi,
                                const int32_t* parent, uint32_t* seg_out, uint32_t* net_cost,
                                int32_t* num_batches, void* stream);
/* fgr_run_host with the Z middles (zmid_out [num_nodes] HOST out, may be NULL). */
FGR_API fgr_status fgr_run_host_ex(fgr_grid* grid, int32_t num_nets, int32_t num_nodes, const int32_t* node_offset,
                                   const int16_t* x, const int16_t* y, const int8_t* pin_lo, const int8_t* pin_hi,
                                   const int32_t* parent, uint32_t* seg_out, int32_t* zmid_out, uint32_t* net_cost,
                                   int32_t* num_batches, void* stream);

/*
 * fgr_overflow — rip-up set extraction after a routing stage (§III-A
 * L398-402 "we first extract the nets to rip up"; §III-G "rewire the
 * nets with violations").  On the grid's current demand, a wire edge is
 * overflowed when demand > capacity, and a net is violating when a committed leg
 * of its route (seg / zmid as written by fgr_route_all(_ex) for `nets`) covers an
 * overflowed edge (R26).
 *   seg [num_nodes], zmid [num_nodes] DEVICE in (zmid may be NULL only while the
 *       grid's pattern is L-only)
 *   violating [num_nets] DEVICE out: 1 / 0 per net
 *   rip_ids [num_nets] DEVICE out: the violating net ids, ascending; *num_rip (host) of them
 *   totals [2] HOST out: overflowed wire edges, sum of (demand - capacity) over them
 * Synchronises `stream`.  Errors: INVALID, CUDA.  Demand is not modified.
 */
FGR_API fgr_status fgr_overflow(fgr_grid* grid, const fgr_nets* nets, const uint32_t* seg, const int32_t* zmid,
                                uint8_t* violating, int32_t* rip_ids, int32_t* num_rip, int64_t* totals, void* stream);

/*
 * fgr_task_graph — the ordered task graph of a set of routing tasks (PAPER.md
 * §III-B, Fig. 6; used for the rip-up tasks, §III-G).
 * Task IDs are the tasks sorted by (HPWL over all tree nodes, net id) (R12);
 * two tasks conflict when their closed bounding boxes share a G-cell (R13); the
 * root task batch is one pass of Algorithm 1 over the task IDs; every
 * conflicting pair is ordered from the root task to the non-root one, else from
 * the smaller task ID to the larger (R27).  The result is acyclic.
 *   tasks [count] DEVICE in: net ids (distinct, any order)
 *   order [count] DEVICE out: net id of task t
 *   is_root [count] DEVICE out: 1 if task t is in the root batch
 *   succ_offset [count+1], succ [capacity] DEVICE out: successors of task t are
 *       succ[succ_offset[t] .. succ_offset[t+1]), task IDs ascending
 *   *num_edges (host) = number of directed edges; RANGE if it exceeds capacity
 *       (succ untouched, succ_offset valid — call again with a larger buffer).
 * Synchronises `stream`.  Errors: INVALID, RANGE, CUDA.
 */
FGR_API fgr_status fgr_task_graph(fgr_grid* grid, const fgr_nets* nets, const int32_t* tasks, int32_t count,
                                  int32_t* order, uint8_t* is_root, int32_t* succ_offset, int32_t* succ,
                                  int64_t capacity, int64_t* num_edges, void* stream);

/* Counters of the last fgr_route_all (for the byte model in DESIGN.md §5). */
typedef struct {
    int64_t refresh_segments;          /* 32-position row/column segments rescanned            */
    int64_t refresh_bytes;             /* algorithmic refresh bytes (D read + cap read + P write) */
    int64_t dp_nets, dp_edges;         /* nets and tree edges routed                            */
    int64_t kernel_launches;           /* kernels launched by the library                       */
    int32_t num_batches, world, rank;
    int32_t exchanged_batches;         /* multi-GPU: batches split across ranks (others routed whole) */
    int32_t graph_mode;                /* batch loop of the call: 0 direct, 1 captured, 2 replayed (fgr_set_graph) */
    int32_t reserved;
} fgr_stats;
FGR_API fgr_status fgr_get_stats(fgr_grid* grid, fgr_stats* out);

/*
 * Per-kernel-class device timing (CUDA events recorded on the caller's stream
 * around every launch of the class while enabled).  Classes:
 *   0 refresh, 1 dp_small (warp per net), 2 dp_large (CTA per net), 3 commit,
 *   4 plan_preprocess, 5 plan_sort (CUB), 6 plan_color, 7 plan_other, 8 exchange (NCCL),
 *   9 hybrid (Z transfer matrices)
 * fgr_profile_read synchronises, then returns the summed milliseconds and the
 * number of launches per class since the last enable, and clears the counters.
 */
#define FGR_PROF_CLASSES 10
FGR_API fgr_status fgr_profile_enable(fgr_grid* grid, int enable);
FGR_API fgr_status fgr_profile_read(fgr_grid* grid, double* ms /* [10] */, int64_t* launches /* [10] */);

#ifdef __cplusplus
}
#endif
#endif /* FASTGR_H */
