// api_grid.cu — grid handle: creation, cost table, demand in/out, errors.
//
// Cost scheme (PAPER.md L556-563 defers to CUGR [3]; our integer reading R1/R2 in
// DESIGN.md §3): ec = len_cost + T_l[clamp(cap - dem, -S, S)], T_l a logistic
// table built once on the host in double and rounded half away from zero.
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "fgr_internal.cuh"

static thread_local char g_err[512] = "";

fgr_status fgr_set_error(fgr_status s, const char* fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return s;
}

fgr_status fgr_cuda_fail(fgr_grid* g, cudaError_t e, const char* where) {
    if (g) g->broken = true;
    if (e == cudaErrorMemoryAllocation) return fgr_set_error(FGR_ERR_OOM, "out of device memory at %s", where);
    return fgr_set_error(FGR_ERR_CUDA, "CUDA error %s (%s) at %s", cudaGetErrorName(e), cudaGetErrorString(e), where);
}

unsigned long long g_scratch_gen = 0;

void fgr_mirrors_free(PlanCache& c) {
    int* ip[6] = {c.h_off, c.h_nlarge, c.h_maxm, c.h_ntwo, c.h_n9, c.h_lsplit};
    for (int* q : ip)
        if (q) cudaFreeHost(q);
    if (c.h_segb) cudaFreeHost(c.h_segb);
    c.h_off = c.h_nlarge = c.h_maxm = c.h_ntwo = c.h_n9 = c.h_lsplit = nullptr;
    c.h_segb = nullptr;
    c.cap = 0;
}

cudaError_t fgr_mirrors_reserve(PlanCache& c, int B) {
    if (c.cap >= B + 1) return cudaSuccess;
    fgr_mirrors_free(c);
    const int cap = B + 1;
    cudaError_t e = cudaMallocHost(&c.h_off, sizeof(int) * cap);
    if (e == cudaSuccess) e = cudaMallocHost(&c.h_nlarge, sizeof(int) * cap);
    if (e == cudaSuccess) e = cudaMallocHost(&c.h_maxm, sizeof(int) * cap);
    if (e == cudaSuccess) e = cudaMallocHost(&c.h_ntwo, sizeof(int) * cap);
    if (e == cudaSuccess) e = cudaMallocHost(&c.h_n9, sizeof(int) * cap);
    if (e == cudaSuccess) e = cudaMallocHost(&c.h_lsplit, sizeof(int) * 5 * cap);
    if (e == cudaSuccess) e = cudaMallocHost(&c.h_segb, sizeof(long long) * cap);
    if (e != cudaSuccess) { fgr_mirrors_free(c); return e; }
    c.cap = cap;
    return cudaSuccess;
}

void* fgr_scratch(Scratch& s, size_t bytes, cudaError_t* err) {
    *err = cudaSuccess;
    if (bytes <= s.bytes && s.p) return s.p;
    g_scratch_gen++;
    if (s.p) cudaFree(s.p);
    s.p = nullptr;
    s.bytes = 0;
    size_t b = bytes < 256 ? 256 : bytes;
    b = b + b / 4;
    *err = cudaMalloc(&s.p, b);
    if (*err != cudaSuccess) { s.p = nullptr; return nullptr; }
    s.bytes = b;
    return s.p;
}

extern "C" FGR_API const char* fgr_last_error(void) { return g_err; }
extern "C" FGR_API const char* fgr_version(void) { return "fastgr-b200 0.1 (sm_100a)"; }

static fgr_status validate_desc(const fgr_grid_desc* d) {
    if (!d) return fgr_set_error(FGR_ERR_INVALID, "desc is NULL");
    if (d->nx < 2 || d->ny < 2 || d->nx > 32767 || d->ny > 32767)
        return fgr_set_error(FGR_ERR_INVALID, "grid dims %dx%d out of [2,32767]", d->nx, d->ny);
    if (d->nlayers < 2 || d->nlayers > FGR_MAXL)
        return fgr_set_error(FGR_ERR_INVALID, "nlayers %d out of [2,16]", d->nlayers);
    if (!d->dir || !d->layer_capacity || !d->via_cost || !d->ovf_weight)
        return fgr_set_error(FGR_ERR_INVALID, "dir/layer_capacity/via_cost/ovf_weight must be non-NULL");
    int nh = 0, nv = 0;
    for (int l = 0; l < d->nlayers; l++) {
        if (d->dir[l] > 1) return fgr_set_error(FGR_ERR_INVALID, "dir[%d]=%d not 0/1", l, d->dir[l]);
        (d->dir[l] ? nv : nh)++;
        if (d->layer_capacity[l] < 0 || d->layer_capacity[l] > 255)
            return fgr_set_error(FGR_ERR_INVALID, "layer_capacity[%d]=%d out of [0,255]", l, d->layer_capacity[l]);
        if (d->ovf_weight[l] < 0) return fgr_set_error(FGR_ERR_INVALID, "ovf_weight[%d] < 0", l);
        if (l + 1 < d->nlayers && d->via_cost[l] < 0) return fgr_set_error(FGR_ERR_INVALID, "via_cost[%d] < 0", l);
    }
    if (nh == 0 || nv == 0) return fgr_set_error(FGR_ERR_INVALID, "need at least one H and one V layer");
    if (d->len_cost < 0) return fgr_set_error(FGR_ERR_INVALID, "len_cost < 0");
    if (d->slack_clamp < 0 || d->slack_clamp > 1024) return fgr_set_error(FGR_ERR_INVALID, "slack_clamp out of [0,1024]");
    if (!std::isfinite(d->logistic_slope)) return fgr_set_error(FGR_ERR_INVALID, "logistic_slope not finite");
    // R19: every leg cost (<= max_ec * max(nx,ny)) must be a finite uint32 cost < 2^31.
    int64_t maxw = 0;
    for (int l = 0; l < d->nlayers; l++) maxw = d->ovf_weight[l] > maxw ? d->ovf_weight[l] : maxw;
    int64_t maxdim = d->nx > d->ny ? d->nx : d->ny;
    if (((int64_t)d->len_cost + maxw) * maxdim >= ((int64_t)1 << 31) - 1)
        return fgr_set_error(FGR_ERR_RANGE, "(len_cost + max ovf_weight) * max(nx,ny) >= 2^31");
    int64_t vsum = 0;
    for (int l = 0; l + 1 < d->nlayers; l++) vsum += d->via_cost[l];
    if (vsum >= ((int64_t)1 << 24)) return fgr_set_error(FGR_ERR_RANGE, "sum of via costs >= 2^24");
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_cost_table(const fgr_grid_desc* d, int64_t* table) {
    fgr_status s = validate_desc(d);
    if (s != FGR_OK) return s;
    int S = d->slack_clamp;
    for (int l = 0; l < d->nlayers; l++)
        for (int k = -S; k <= S; k++)
            table[(int64_t)l * (2 * S + 1) + (k + S)] =
                std::llround((double)d->ovf_weight[l] / (1.0 + std::exp(d->logistic_slope * (double)k)));
    return FGR_OK;
}

// dense [L][ny][nx] <-> sector layouts
__global__ void k_dense_to_sector_u8(GridView g, const uint8_t* dense, const int32_t* layer_cap, uint8_t* CH,
                                     uint8_t* CV) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    int64_t n = (int64_t)g.L * g.ny * g.nx;
    if (i >= n) return;
    int x = (int)(i % g.nx);
    int y = (int)((i / g.nx) % g.ny);
    int l = (int)(i / ((int64_t)g.nx * g.ny));
    uint8_t c = dense ? dense[i] : (uint8_t)layer_cap[l];
    if (g.dir[l] == 0) CH[((int64_t)y * g.nx + x) * g.h.W + g.slot[l]] = c;
    else CV[((int64_t)x * g.ny + y) * g.v.W + g.slot[l]] = c;
}

__global__ void k_demand_set(GridView g, const int32_t* dense) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    int64_t n = (int64_t)g.L * g.ny * g.nx;
    if (i >= n) return;
    int x = (int)(i % g.nx);
    int y = (int)((i / g.nx) % g.ny);
    int l = (int)(i / ((int64_t)g.nx * g.ny));
    if (g.dir[l] == 0) g.h.D[((int64_t)y * g.nx + x) * g.h.W + g.slot[l]] = (x == g.nx - 1) ? 0 : dense[i];
    else g.v.D[((int64_t)x * g.ny + y) * g.v.W + g.slot[l]] = (y == g.ny - 1) ? 0 : dense[i];
}

__global__ void k_demand_get(GridView g, int32_t* dense) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    int64_t n = (int64_t)g.L * g.ny * g.nx;
    if (i >= n) return;
    int x = (int)(i % g.nx);
    int y = (int)((i / g.nx) % g.ny);
    int l = (int)(i / ((int64_t)g.nx * g.ny));
    if (g.dir[l] == 0) dense[i] = (x == g.nx - 1) ? 0 : g.h.D[((int64_t)y * g.nx + x) * g.h.W + g.slot[l]];
    else dense[i] = (y == g.ny - 1) ? 0 : g.v.D[((int64_t)x * g.ny + y) * g.v.W + g.slot[l]];
}

static int pow2_at_least4(int n) {
    int w = 4;
    while (w < n) w *= 2;
    return w;
}

static size_t align256(size_t b) { return (b + 255) & ~(size_t)255; }

extern "C" FGR_API fgr_status fgr_grid_create(const fgr_grid_desc* d, int device, void* stream, fgr_grid** out) {
    if (!out) return fgr_set_error(FGR_ERR_INVALID, "out is NULL");
    *out = nullptr;
    fgr_status s = validate_desc(d);
    if (s != FGR_OK) return s;
    cudaError_t e = cudaSetDevice(device);
    if (e != cudaSuccess) return fgr_cuda_fail(nullptr, e, "cudaSetDevice");
    cudaStream_t st = (cudaStream_t)stream;
    fgr_grid* g = new fgr_grid();
    g->device = device;
    g->nx = d->nx; g->ny = d->ny; g->L = d->nlayers; g->S = d->slack_clamp; g->len_cost = d->len_cost;
    g->slope = d->logistic_slope;
    GridView& v = g->view;
    memset(&v, 0, sizeof(v));
    for (int l = 0; l < g->L; l++) {
        g->dir[l] = d->dir[l];
        g->layer_capacity[l] = d->layer_capacity[l];
        g->ovf_weight[l] = d->ovf_weight[l];
        g->via_cost[l] = (l + 1 < g->L) ? d->via_cost[l] : 0;
        int dd = d->dir[l];
        int sl = dd ? g->nV++ : g->nH++;
        v.dir[l] = (uint8_t)dd;
        v.slot[l] = (uint8_t)sl;
        v.layer_of_slot[dd][sl] = (uint8_t)l;
    }
    v.viapre[0] = 0;
    for (int l = 0; l < g->L; l++) v.viapre[l + 1] = v.viapre[l] + (uint32_t)g->via_cost[l];
    g->WH = pow2_at_least4(g->nH);
    g->WV = pow2_at_least4(g->nV);
    v.nx = g->nx; v.ny = g->ny; v.L = g->L; v.S = g->S; v.len_cost = g->len_cost;
    DirView& h = v.h;
    DirView& w = v.v;
    h.len = g->nx; h.lines = g->ny; h.W = g->WH; h.cnt = g->nH; h.nseg = (g->nx + FGR_SEG - 1) / FGR_SEG;
    w.len = g->ny; w.lines = g->nx; w.W = g->WV; w.cnt = g->nV; w.nseg = (g->ny + FGR_SEG - 1) / FGR_SEG;
    h.seg_base = 0; w.seg_base = h.lines * h.nseg;
    h.line_base = 0; w.line_base = h.lines;
    g->total_segs = h.lines * h.nseg + w.lines * w.nseg;
    size_t cells = (size_t)g->nx * g->ny;
    size_t bH = cells * g->WH, bV = cells * g->WV;
    size_t sH = (size_t)h.lines * h.nseg * g->WH, sV = (size_t)w.lines * w.nseg * g->WV;
    size_t sizes[] = {bH * 4, bV * 4, bH, bV, bH * 4, bV * 4, sH * 4, sV * 4, sH * 4, sV * 4,
                      (size_t)g->total_segs, (size_t)(g->nx + g->ny), (size_t)(g->nx + g->ny) * 4};
    size_t total = 0;
    for (size_t z : sizes) total += align256(z);
    e = cudaMalloc(&g->mem, total);
    if (e != cudaSuccess) { delete g; return fgr_cuda_fail(nullptr, e, "cudaMalloc(grid)"); }
    g->mem_bytes = total;
    char* p = (char*)g->mem;
    void* ptrs[13];
    for (int i = 0; i < 13; i++) { ptrs[i] = p; p += align256(sizes[i]); }
    h.D = (int32_t*)ptrs[0]; w.D = (int32_t*)ptrs[1];
    h.C = (const uint8_t*)ptrs[2]; w.C = (const uint8_t*)ptrs[3];
    h.P = (uint32_t*)ptrs[4]; w.P = (uint32_t*)ptrs[5];
    h.ST = (uint32_t*)ptrs[6]; w.ST = (uint32_t*)ptrs[7];
    h.SB = (uint32_t*)ptrs[8]; w.SB = (uint32_t*)ptrs[9];
    v.dseg = (uint8_t*)ptrs[10]; v.dline = (uint8_t*)ptrs[11]; v.linedone = (uint32_t*)ptrs[12];
    // lists, counters, table
    size_t tab = (size_t)g->L * (2 * g->S + 1);
    int32_t* htab = (int32_t*)malloc(tab * sizeof(int32_t));
    for (int l = 0; l < g->L; l++)
        for (int k = -g->S; k <= g->S; k++)
            htab[(size_t)l * (2 * g->S + 1) + (k + g->S)] =
                (int32_t)std::llround((double)g->ovf_weight[l] / (1.0 + std::exp(g->slope * (double)k)));
    bool ok = cudaMalloc(&g->d_table, tab * sizeof(int32_t)) == cudaSuccess &&
              cudaMalloc(&g->d_stats, 4 * sizeof(unsigned long long)) == cudaSuccess;
    if (!ok) { free(htab); fgr_grid_destroy(g); return fgr_set_error(FGR_ERR_OOM, "out of device memory (grid)"); }
    v.table = g->d_table;
    v.stats = g->d_stats;
    cudaMemcpyAsync(g->d_table, htab, tab * sizeof(int32_t), cudaMemcpyHostToDevice, st);
    cudaMemsetAsync(g->mem, 0, total, st);
    cudaMemsetAsync(g->d_stats, 0, 4 * sizeof(unsigned long long), st);
    int32_t hcap[FGR_MAXL];
    for (int l = 0; l < g->L; l++) hcap[l] = g->layer_capacity[l];
    int32_t* dcap = nullptr;
    cudaMalloc(&dcap, sizeof(hcap));
    cudaMemcpyAsync(dcap, hcap, sizeof(hcap), cudaMemcpyHostToDevice, st);
    int64_t n = (int64_t)g->L * cells;
    k_dense_to_sector_u8<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(v, d->edge_capacity, dcap, (uint8_t*)h.C,
                                                                         (uint8_t*)w.C);
    e = cudaStreamSynchronize(st);
    cudaFree(dcap);
    free(htab);
    if (e == cudaSuccess) e = cudaGetLastError();
    if (e != cudaSuccess) { fgr_grid_destroy(g); return fgr_cuda_fail(nullptr, e, "grid init"); }
    g->full_dirty = true;
    bool sok = cudaEventCreateWithFlags(&g->ev_fork, cudaEventDisableTiming) == cudaSuccess;
    for (int i = 0; i < FGR_SIDE_STREAMS && sok; i++)
        sok = cudaStreamCreateWithFlags(&g->side[i], cudaStreamNonBlocking) == cudaSuccess &&
              cudaEventCreateWithFlags(&g->ev_join[i], cudaEventDisableTiming) == cudaSuccess;
    if (!sok) {
        fgr_grid_destroy(g);
        return fgr_set_error(FGR_ERR_CUDA, "stream/event creation failed");
    }
    cudaDeviceGetAttribute(&g->max_smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, device);
    cudaDeviceGetAttribute(&g->num_sms, cudaDevAttrMultiProcessorCount, device);
    g->stats.world = 1;
    *out = g;
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_grid_destroy(fgr_grid* g) {
    if (!g) return FGR_OK;
    cudaSetDevice(g->device);
    if (g->rg.exec) cudaGraphExecDestroy(g->rg.exec);
    if (g->rg.cap) cudaStreamDestroy(g->rg.cap);
    if (g->comm) ncclCommDestroy(g->comm);
    cudaFree(g->mem);
    cudaFree(g->d_table);
    cudaFree(g->d_stats);
    for (auto& s : g->s_plan) cudaFree(s.p);
    for (auto& s : g->s_rec) cudaFree(s.p);
    cudaFree(g->s_prep.p);
    for (auto& s : g->s_hyb) cudaFree(s.p);
    for (auto& s : g->s_rip) cudaFree(s.p);
    for (auto e : g->prof.pool) cudaEventDestroy(e);
    for (int i = 0; i < FGR_SIDE_STREAMS; i++) {
        if (g->side[i]) cudaStreamDestroy(g->side[i]);
        if (g->ev_join[i]) cudaEventDestroy(g->ev_join[i]);
    }
    if (g->ev_fork) cudaEventDestroy(g->ev_fork);
    fgr_mirrors_free(g->cache);
    delete g;
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_grid_set_demand(fgr_grid* g, const int32_t* demand, void* stream) {
    if (!g) return fgr_set_error(FGR_ERR_INVALID, "grid is NULL");
    if (g->broken) return fgr_set_error(FGR_ERR_STATE, "grid unusable after an earlier CUDA/NCCL error");
    cudaStream_t st = (cudaStream_t)stream;
    FGR_CHECK_CUDA(g, cudaSetDevice(g->device));
    const GridView& v = g->view;
    if (!demand) {
        FGR_CHECK_CUDA(g, cudaMemsetAsync(v.h.D, 0, (size_t)g->nx * g->ny * g->WH * 4, st));
        FGR_CHECK_CUDA(g, cudaMemsetAsync(v.v.D, 0, (size_t)g->nx * g->ny * g->WV * 4, st));
    } else {
        int64_t n = (int64_t)g->L * g->nx * g->ny;
        k_demand_set<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(v, demand);
        FGR_CHECK_CUDA(g, cudaGetLastError());
    }
    g->full_dirty = true;
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_grid_get_demand(fgr_grid* g, int32_t* demand, void* stream) {
    if (!g || !demand) return fgr_set_error(FGR_ERR_INVALID, "grid or demand is NULL");
    if (g->broken) return fgr_set_error(FGR_ERR_STATE, "grid unusable after an earlier CUDA/NCCL error");
    cudaStream_t st = (cudaStream_t)stream;
    FGR_CHECK_CUDA(g, cudaSetDevice(g->device));
    int64_t n = (int64_t)g->L * g->nx * g->ny;
    k_demand_get<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(g->view, demand);
    FGR_CHECK_CUDA(g, cudaGetLastError());
    return FGR_OK;
}

int fgr_prof_begin(fgr_grid* g, int cls, cudaStream_t st) {
    Profiler& p = g->prof;
    if (!p.on) return -1;
    if (p.used * 2 + 2 > p.pool.size()) {
        for (int i = 0; i < 256; i++) {
            cudaEvent_t e;
            if (cudaEventCreate(&e) != cudaSuccess) return -1;
            p.pool.push_back(e);
        }
    }
    const int slot = (int)p.used++;
    if (p.cls.size() < p.used) p.cls.resize(p.used);
    p.cls[slot] = cls;
    cudaEventRecord(p.pool[2 * slot], st);
    return slot;
}

void fgr_prof_end(fgr_grid* g, int slot, cudaStream_t st) {
    if (slot < 0) return;
    cudaEventRecord(g->prof.pool[2 * slot + 1], st);
}

extern "C" FGR_API fgr_status fgr_profile_enable(fgr_grid* g, int enable) {
    if (!g) return fgr_set_error(FGR_ERR_INVALID, "grid is NULL");
    g->prof.on = enable != 0;
    g->prof.used = 0;
    for (int i = 0; i < FGR_PROF_CLASSES; i++) { g->prof.ms[i] = 0; g->prof.launches[i] = 0; }
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_profile_read(fgr_grid* g, double* ms, int64_t* launches) {
    if (!g || !ms || !launches) return fgr_set_error(FGR_ERR_INVALID, "NULL argument");
    Profiler& p = g->prof;
    FGR_CHECK_CUDA(g, cudaSetDevice(g->device));
    for (size_t i = 0; i < p.used; i++) {
        FGR_CHECK_CUDA(g, cudaEventSynchronize(p.pool[2 * i + 1]));
        float t = 0;
        FGR_CHECK_CUDA(g, cudaEventElapsedTime(&t, p.pool[2 * i], p.pool[2 * i + 1]));
        p.ms[p.cls[i]] += t;
        p.launches[p.cls[i]]++;
    }
    p.used = 0;
    for (int i = 0; i < FGR_PROF_CLASSES; i++) {
        ms[i] = p.ms[i];
        launches[i] = p.launches[i];
        p.ms[i] = 0;
        p.launches[i] = 0;
    }
    return FGR_OK;
}

extern "C" FGR_API fgr_status fgr_get_stats(fgr_grid* g, fgr_stats* out) {
    if (!g || !out) return fgr_set_error(FGR_ERR_INVALID, "grid or out is NULL");
    if (g->broken) return fgr_set_error(FGR_ERR_STATE, "grid unusable after an earlier CUDA/NCCL error");
    unsigned long long hs[4];
    FGR_CHECK_CUDA(g, cudaMemcpy(hs, g->d_stats, sizeof(hs), cudaMemcpyDeviceToHost));
    *out = g->stats;
    out->refresh_segments = (int64_t)(hs[0] + hs[1]);
    // per refreshed segment: 32 positions x (demand int32 read + capacity byte read + prefix uint32 write)
    out->refresh_bytes = (int64_t)(hs[0] * 32ull * 9ull * (unsigned long long)g->WH +
                                   hs[1] * 32ull * 9ull * (unsigned long long)g->WV);
    return FGR_OK;
}
