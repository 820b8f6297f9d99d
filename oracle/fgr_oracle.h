/*
 * fgr_oracle.h — plain, slow, single-threaded CPU oracle for batched 3-D
 * L-shape pattern routing with layer assignment (FastGR, §III-C/D).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.  It
 * shares no code, header, table or constant generator with the CUDA path
 * (paper_conf_date_liulzclly22_b200/), and never includes include/fastgr.h.
 *
 * Layouts (plain, dense):
 *   demand / edge_capacity : [L][ny][nx].  For an H layer, entry (y,x) is the
 *   wire edge (x,y)-(x+1,y) (x = nx-1 unused); for a V layer, entry (y,x) is the
 *   wire edge (x,y)-(x,y+1) (y = ny-1 unused).
 *   seg[node] (node = global node index of the child endpoint of a tree edge):
 *   bend | ls<<8 | lt<<16 | straight<<24; roots get 0xFFFFFFFF.  bend 0/1 = the
 *   two L shapes; with hybrid patterns also 2 = Z HVH, 3 = Z VHV, whose middle
 *   coordinate (xm for HVH, ym for VHV) and middle layer lb are in
 *   zmid[node] = mid | lb << 16 (-1 for every non-Z edge).
 */
#ifndef FGR_ORACLE_H
#define FGR_ORACLE_H
#include <stdint.h>

typedef struct {
    int32_t nx, ny, nlayers;
    const uint8_t* dir;             /* [L] 0 = H, 1 = V                                  */
    const int32_t* layer_capacity;  /* [L]                                               */
    const uint8_t* edge_capacity;   /* [L][ny][nx] or NULL                               */
    int32_t len_cost;               /* wirelength cost per unit edge                     */
    const int32_t* via_cost;        /* [L-1] cost of one via hop k -> k+1                */
    const int32_t* ovf_weight;      /* [L] logistic weight W_l                           */
    double logistic_slope;
    int32_t slack_clamp;
} orc_grid;

typedef struct {
    int32_t num_nets;
    const int32_t* node_offset;     /* [N+1] */
    const int16_t* x;
    const int16_t* y;
    const int8_t* pin_lo;
    const int8_t* pin_hi;
    const int32_t* parent;          /* net-local; parent[i] < i; -1 at local 0 */
} orc_nets;

/* Hybrid L+Z selection (§III-F and §IV-D):
 * bent tree edges with hybrid_lo <= |dx|+|dy| <= hybrid_hi take the hybrid
 * patterns (the paper's "medium" two-pin nets, t1 = 100, t2 = 500); all other
 * edges the L patterns.  NULL pattern (or lo > hi) = L only (FastGRL). */
typedef struct {
    int32_t hybrid_lo, hybrid_hi;
} orc_pattern;

#define ORC_OK 0
#define ORC_INVALID 1
#define ORC_RANGE 2

int orc_cost_table(const orc_grid* g, int64_t* table /* [L][2S+1] */);
int orc_validate(const orc_grid* g, const orc_nets* n, int32_t* bad_net);
int orc_plan(const orc_grid* g, const orc_nets* n, int32_t* batch_of_net, int32_t* num_batches);
int orc_route_net(const orc_grid* g, const orc_nets* n, int32_t net, const int32_t* demand,
                  uint32_t* seg /* [num_nodes] global */, uint32_t* net_cost);
int orc_commit_net(const orc_grid* g, const orc_nets* n, int32_t net, const uint32_t* seg, int32_t* demand);
int orc_route(const orc_grid* g, const orc_nets* n, const int32_t* batch_of_net, int32_t num_batches,
              int32_t* demand, uint32_t* seg, uint32_t* net_cost, int sequential_within_batch,
              uint64_t* batch_hash /* [num_batches] or NULL */);
int orc_recost_net(const orc_grid* g, const orc_nets* n, int32_t net, const int32_t* demand,
                   const uint32_t* seg, uint64_t* cost);

int orc_route_net_ex(const orc_grid* g, const orc_nets* n, int32_t net, const int32_t* demand,
                     uint32_t* seg, uint32_t* net_cost, const orc_pattern* pat, int32_t* zmid);
int orc_commit_net_ex(const orc_grid* g, const orc_nets* n, int32_t net, const uint32_t* seg, const int32_t* zmid,
                      int32_t* demand);
int orc_route_ex(const orc_grid* g, const orc_nets* n, const int32_t* batch_of_net, int32_t num_batches,
                 int32_t* demand, uint32_t* seg, uint32_t* net_cost, int sequential_within_batch,
                 uint64_t* batch_hash, const orc_pattern* pat, int32_t* zmid);
int orc_recost_net_ex(const orc_grid* g, const orc_nets* n, int32_t net, const int32_t* demand,
                      const uint32_t* seg, const int32_t* zmid, uint64_t* cost);
/* rip-up set extraction (violating nets) and overflow totals on a final demand */
int orc_overflow(const orc_grid* g, const orc_nets* n, const uint32_t* seg, const int32_t* zmid,
                 const int32_t* demand, uint8_t* violating, int64_t* totals /* [2] */);
/* ordered task graph of a task set (net ids): task order, root batch, successor CSR */
int orc_task_graph(const orc_grid* g, const orc_nets* n, const int32_t* tasks, int32_t count, int32_t* order,
                   uint8_t* is_root, int32_t* succ_off, int32_t* succ, int64_t cap, int64_t* num_edges);

#endif
