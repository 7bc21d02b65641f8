// api.cu -- the C ABI of libdbc (include/dbc.h): context, HBM arena, root
// sharding, batch flow, error model.  Every compute step runs in the kernels of
// static_brandes.cu / update.cu / graph.cu; this file only validates,
// allocates, launches and copies.
#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <thread>
#include <unordered_set>
#include <vector>

#include <dlfcn.h>
#include <nccl.h>  // types only: NCCL is loaded at run time (dlopen), never linked

#include "dbc.h"
#include "dbc_internal.cuh"
#include "graph_ops.h"

using namespace dbc;

// NCCL entry points, resolved from libnccl.so.2 at first use -- the copy
// PyTorch already loaded into the process when there is one (same NCCL as its
// process groups), else the system's.
struct NcclApi {
    bool ok = false;
    std::string why;
    ncclResult_t (*get_unique_id)(ncclUniqueId *) = nullptr;
    ncclResult_t (*comm_init_rank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*all_reduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                               cudaStream_t) = nullptr;
    ncclResult_t (*comm_destroy)(ncclComm_t) = nullptr;
    const char *(*error_string)(ncclResult_t) = nullptr;
};
static NcclApi &nccl_api() {
    static NcclApi api = [] {
        NcclApi a;
        void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) {
            const char *e = dlerror();
            a.why = e ? e : "libnccl.so.2 not found";
            return a;
        }
        a.get_unique_id = (decltype(a.get_unique_id))dlsym(h, "ncclGetUniqueId");
        a.comm_init_rank = (decltype(a.comm_init_rank))dlsym(h, "ncclCommInitRank");
        a.all_reduce = (decltype(a.all_reduce))dlsym(h, "ncclAllReduce");
        a.comm_destroy = (decltype(a.comm_destroy))dlsym(h, "ncclCommDestroy");
        a.error_string = (decltype(a.error_string))dlsym(h, "ncclGetErrorString");
        a.ok = a.get_unique_id && a.comm_init_rank && a.all_reduce && a.comm_destroy && a.error_string;
        if (!a.ok) a.why = "libnccl.so.2 lacks an entry point";
        return a;
    }();
    return api;
}

struct dbc_ctx {
    int device = 0, rank = 0, world = 1;
    uint32_t flags = 0;
    int32_t n = 0;
    int64_t nnz = 0, nnz0 = 0, col_cap = 0;
    int64_t deleted = 0;  // edges deleted (tombstones in the rows)
    int64_t edge_cap = 0, inserted = 0;
    int32_t k = 0, k_loc = 0;
    std::vector<int32_t> roots_local;        // internal vertex ids of the local roots
    std::vector<int32_t> perm, iperm;        // external -> internal id, internal -> external
    int32_t *perm_d = nullptr;               // device copy of perm
    double *bc_ext = nullptr;                // BC partial in external order (for callers)
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    int workers = 0;
    int block = 512;   // threads per update worker CTA (512, 256 or 128)
    bool ub2 = false;  // 512-thread CTAs built for two per SM (update_512x2)
    bool lowdeg = false;  // max degree <= 32 (mesh-like graphs)
    int64_t maxdeg0 = 0;  // max degree of the initial graph
    int hd_min = 1024, hd_block = 512;  // helped down levels (update.cu)
    int he_entries = 8192, he_min = 3;   // helped flattened passes (update.cu)
    int busy_help = 4;                   // blocks a busy worker takes at a level boundary
                                         // (re-tuned after the counter lanes, DESIGN.md Sec. 9:
                                         // 1 -> 4 and 4096 -> 8192 entries, R-MAT 16 -8%)
    int busy_min = 32;                   // ... of passes of at least this many blocks
    int dl_min = 16 * 4096;              // entry-balanced long rows of a down level from this many entries
    int wide_inlane = -1;                // up levels of <= this many items per thread: short rows in-lane
    int sblock = 256, sworkers = 0;  // static kernel: its own CTA width and grid
    int lean_workers = 0;            // update_lean.cu worker CTAs (one job per insertion)
    bool lean_on = true;             // per-insertion jobs on update_lean.cu (else update.cu)
    int64_t lean_max = 1;            // merged batches of <= this many insertions also run there
    int lean_short = 4;              // level-2 shortcut threshold (rows > lean_short x deg(root))
    int lean_block = 128;            // threads per update_lean.cu CTA
    int lean_narrow = 0;             // > 0: 128-thread workers for multi-insertion launches (meshes)
    int lean_pair = 0;               // > 0: 512-thread 64-register workers (two per SM) for
                                     //      multi-insertion launches on hub graphs
    void *lean_board = nullptr;      // its help board (one entry per worker)
    size_t nscratch = 0;             // worker scratch sets allocated
    // heavy lanes: the slowest root chains of the previous batch run on
    // 2x-wide CTAs (hblock threads) on a high-priority stream
    int hblock = 512, heavy_cap = 0;
    cudaStream_t hstream = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    int32_t *slots_d = nullptr;
    std::vector<double> root_ms;   // chain time per local slot, last Mode-A launch
    HelpBoard help{};              // cooperative help board (Mode A)
    bool help_on = true;
    bool prof_pending = false;
    int nsm = 148;
    bool have_state = false;
    uint64_t epoch_used = 0;

    // graph double buffer
    int32_t *rp[2] = {nullptr, nullptr};
    int32_t *col[2] = {nullptr, nullptr};
    int32_t *scol[2] = {nullptr, nullptr};  // rows sorted by neighbour id
    int cur = 0;
    AppendBufs ab{};
    int32_t *bu = nullptr, *bv = nullptr;  // host-API batch staging

    // state
    int32_t *d = nullptr;    // [k_loc][n]
    double2 *sd = nullptr;   // [k_loc][n] (sigma, delta)
    uint32_t *l2mask = nullptr;  // [k_loc][n] level-2 predecessor masks
    int32_t *mask_ds = nullptr;  // [k_loc]
    double *bc = nullptr;
    int32_t *roots_d = nullptr;

    Scratch ws{};
    int32_t *next_slot = nullptr;
    bool lean_clean = false;          // next_slot[0..4] zero: left so by the per-insertion kernel's last CTA
    unsigned long long *stats = nullptr;
    int32_t *err = nullptr;
    unsigned long long *root_prof = nullptr;  // [k_loc][4], filled when profiling is on
    bool prof_on = false;
    int32_t *esrc = nullptr, *etag = nullptr;  // edge-parallel mode: entry source / insertion index
    double *eodel = nullptr;                   // edge-parallel mode: old delta per worker and vertex
    int eworkers = 0;
    long long *scen = nullptr;  // scenario log [insertion][k_loc] of the last insert call
    int64_t scen_cap = 0;       // insertions it holds (0: logging off)
    int64_t scen_alloc = 0;     // insertions the allocation holds
    int64_t scen_last = 0;      // insertions logged by the last insert call

    std::vector<void *> allocs;
    int64_t bytes = 0;
    dbc_alloc_fn dev_alloc = nullptr;  // caller's device allocator (nullable)
    dbc_free_fn dev_free = nullptr;
    void *alloc_user = nullptr;
    dbc_tuning tune{};                 // launch configuration (dbc_tuning_default: automatic)
    ncclComm_t comm = nullptr;         // BC all-reduce across ranks (opt.nccl_id)
    dbc_reduce_fn reduce = nullptr;    // ... or the caller's callback (opt.reduce)
    void *reduce_user = nullptr;

    // Host copy of the adjacency in caller ids: the original rows sorted, plus
    // the edges inserted / original edges deleted since (key min << 32 | max).
    // Host-array batches are validated against it (no device round trip).
    std::vector<int64_t> h_rp;
    std::vector<int32_t> h_scol;
    std::unordered_set<uint64_t> h_ins, h_del;
    int32_t *h_pin = nullptr;       // pinned staging of device-array batches for the host copy
    cudaEvent_t ev_prof = nullptr;  // recorded after a batch whose chain times are pending
    cudaEvent_t ev[10] = {};  // [0..3]/[6..9]: insert-call sets A/B, [4..5]: static
    int evset = 0;            // set of the most recent insert call (0 -> ev[0..3], 1 -> ev[6..9])
    bool ev_ok = false;
    dbc_timings tm{};
    bool tm_pending = false, tm_static = false;
    unsigned long long bytes_base = 0;

    std::string msg;
};

static thread_local std::string g_create_msg;

static dbc_status fail(dbc_ctx *c, dbc_status s, const char *fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    if (c)
        c->msg = buf;
    else
        g_create_msg = buf;
    return s;
}

#define CK(call)                                                                           \
    do {                                                                                   \
        cudaError_t e_ = (call);                                                           \
        if (e_ != cudaSuccess)                                                             \
            return fail(c, DBC_ECUDA, "%s: %s (%s:%d)", #call, cudaGetErrorString(e_),     \
                        __FILE__, __LINE__);                                               \
    } while (0)

template <class T>
static dbc_status dalloc(dbc_ctx *c, T **p, size_t count) {
    size_t b = std::max<size_t>(count, 1) * sizeof(T);
    void *q = nullptr;
    if (c->dev_alloc) {  // the caller's allocator (e.g. torch's caching allocator)
        q = c->dev_alloc(b, c->alloc_user);
        if (!q) return fail(c, DBC_ENOMEM, "dev_alloc(%zu bytes) failed", b);
    } else {
        cudaError_t e = cudaMalloc(&q, b);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(c, DBC_ENOMEM, "cudaMalloc(%zu bytes) failed: %s", b, cudaGetErrorString(e));
        }
    }
    c->allocs.push_back(q);
    c->bytes += (int64_t)b;
    *p = (T *)q;
    return DBC_OK;
}

// A temporary device buffer (not kept by the context): the caller frees it with dfree.
static void *talloc(dbc_ctx *c, size_t b) {
    b = std::max<size_t>(b, 1);
    void *q = nullptr;
    if (c->dev_alloc) return c->dev_alloc(b, c->alloc_user);
    if (cudaMalloc(&q, b) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    return q;
}

static void dfree(dbc_ctx *c, void *p) {
    if (!p) return;
    if (c->dev_free)
        c->dev_free(p, c->alloc_user);
    else
        cudaFree(p);
}

#define TRY(x)                          \
    do {                                \
        dbc_status s_ = (x);            \
        if (s_ != DBC_OK) return s_;    \
    } while (0)

extern "C" {

void dbc_options_default(dbc_options *opt) {
    if (!opt) return;
    std::memset(opt, 0, sizeof(*opt));
    opt->world = 1;
}

void dbc_tuning_default(dbc_tuning *t) {
    if (!t) return;
    std::memset(t, 0, sizeof(*t));
    t->update_block = t->update_pair = t->static_block = t->window = t->heavy_cap = -1;
    t->help_down_min = t->help_down_block = t->help_entries = t->help_min_blocks = -1;
    t->busy_help = t->busy_min = t->down_long_min = t->wide_inlane = -1;
    t->lean_block = t->lean_workers = t->lean_max_batch = t->lean_short = t->trace_slot = -1;
    t->static_ms = t->static_groups = t->static_chunk = t->static_width = -1;
    t->heavy_factor = 0.0f;
}

dbc_status dbc_nccl_unique_id(void *out) {
    if (!out) return DBC_EINVAL;
    NcclApi &nc = nccl_api();
    if (!nc.ok) {
        g_create_msg = "NCCL unavailable: " + nc.why;
        return DBC_ENCCL;
    }
    ncclUniqueId id;
    const ncclResult_t r = nc.get_unique_id(&id);
    if (r != ncclSuccess) {
        g_create_msg = std::string("ncclGetUniqueId: ") + nc.error_string(r);
        return DBC_ENCCL;
    }
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    std::memcpy(out, &id, sizeof id);
    return DBC_OK;
}

int32_t dbc_abi_version(void) { return DBC_ABI_VERSION; }

const char *dbc_strerror(dbc_status s) {
    switch (s) {
        case DBC_OK: return "ok";
        case DBC_EINVAL: return "invalid argument";
        case DBC_ENOMEM: return "out of memory";
        case DBC_ECUDA: return "CUDA error";
        case DBC_ENCCL: return "collective error";
        case DBC_ESTATE: return "call out of order";
        case DBC_EEDGE: return "invalid edge in batch";
        case DBC_ECAPACITY: return "inserted-edge capacity exhausted";
        case DBC_ENUMERIC: return "shortest-path count overflowed";
    }
    return "unknown status";
}

const char *dbc_last_error(const dbc_ctx *c) { return c ? c->msg.c_str() : g_create_msg.c_str(); }

void dbc_destroy(dbc_ctx *c) {
    if (!c) return;
    cudaSetDevice(c->device);
    if (c->stream) cudaStreamSynchronize(c->stream);
    if (c->comm) nccl_api().comm_destroy(c->comm);
    for (void *p : c->allocs) dfree(c, p);
    if (c->ev_ok)
        for (auto &e : c->ev) cudaEventDestroy(e);
    if (c->ev_fork) cudaEventDestroy(c->ev_fork);
    if (c->ev_prof) cudaEventDestroy(c->ev_prof);
    if (c->h_pin) cudaFreeHost(c->h_pin);
    if (c->ev_join) cudaEventDestroy(c->ev_join);
    if (c->hstream) cudaStreamDestroy(c->hstream);
    if (c->own_stream && c->stream) cudaStreamDestroy(c->stream);
    delete c;
}

}  // extern "C"

// Host CSR validation: symmetric, no self loops, no duplicate entries.
static bool validate_csr(int32_t n, const int64_t *rp, const int32_t *col, std::string &why,
                         std::vector<int32_t> *sorted_out) {
    if (rp[0] != 0) { why = "row_ptr[0] != 0"; return false; }
    for (int32_t v = 0; v < n; ++v)
        if (rp[v + 1] < rp[v]) { why = "row_ptr not non-decreasing"; return false; }
    const int64_t nnz = rp[n];
    for (int64_t j = 0; j < nnz; ++j)
        if (col[j] < 0 || col[j] >= n) { why = "col entry out of range"; return false; }
    // sorted copies of every row, then per-entry reverse lookup
    std::vector<int32_t> srt(col, col + nnz);
    unsigned nt = std::max(1u, std::min(32u, std::thread::hardware_concurrency()));
    std::vector<std::string> whys(nt);
    std::vector<int> ok(nt, 1);
    auto sort_rows = [&](unsigned t) {
        for (int64_t v = t; v < n; v += nt) std::sort(srt.begin() + rp[v], srt.begin() + rp[v + 1]);
    };
    auto check_rows = [&](unsigned t) {
        for (int64_t v = t; v < n && ok[t]; v += nt) {
            for (int64_t j = rp[v]; j < rp[v + 1]; ++j) {
                const int32_t y = srt[j];
                if (y == v) { ok[t] = 0; whys[t] = "self loop at vertex " + std::to_string(v); break; }
                if (j > rp[v] && srt[j - 1] == y) {
                    ok[t] = 0; whys[t] = "duplicate entry in row " + std::to_string(v); break;
                }
                if (!std::binary_search(srt.begin() + rp[y], srt.begin() + rp[y + 1], (int32_t)v)) {
                    ok[t] = 0;
                    whys[t] = "CSR not symmetric: " + std::to_string(v) + "->" + std::to_string(y);
                    break;
                }
            }
        }
    };
    {
        std::vector<std::thread> th;
        for (unsigned t = 0; t < nt; ++t) th.emplace_back(sort_rows, t);
        for (auto &x : th) x.join();
    }
    {
        std::vector<std::thread> th;
        for (unsigned t = 0; t < nt; ++t) th.emplace_back(check_rows, t);
        for (auto &x : th) x.join();
    }
    for (unsigned t = 0; t < nt; ++t)
        if (!ok[t]) { why = whys[t]; return false; }
    if (sorted_out) *sorted_out = std::move(srt);
    return true;
}

// Locality relabelling (internal only): vertices in BFS order per component,
// components started from a minimum-degree vertex, isolated vertices last.
// Neighbours with nearby ids make the random d / sigma gathers of a level share
// sectors and cache lines.  Row entry order is preserved (canonical order of
// the sums, R5), so results are bit-identical to the unrelabelled run.
static void bfs_order(int32_t n, const int64_t *rp, const int32_t *col, std::vector<int32_t> &perm,
                      std::vector<int32_t> &iperm) {
    std::vector<int32_t> byDeg;
    byDeg.reserve(n);
    int64_t maxdeg = 0;
    for (int32_t v = 0; v < n; ++v) maxdeg = std::max<int64_t>(maxdeg, rp[v + 1] - rp[v]);
    {  // counting sort of non-isolated vertices by degree
        std::vector<int64_t> cnt((size_t)maxdeg + 2, 0);
        for (int32_t v = 0; v < n; ++v) cnt[(size_t)(rp[v + 1] - rp[v])]++;
        std::vector<int64_t> pos((size_t)maxdeg + 2, 0);
        for (int64_t d = 1; d <= maxdeg; ++d) pos[d + 1] = pos[d] + cnt[d];
        byDeg.assign((size_t)(n - cnt[0]), 0);
        for (int32_t v = 0; v < n; ++v) {
            const int64_t d = rp[v + 1] - rp[v];
            if (d > 0) byDeg[(size_t)pos[d]++] = v;
        }
    }
    perm.assign(n, -1);
    iperm.clear();
    iperm.reserve(n);
    for (int32_t s0 : byDeg) {
        if (perm[s0] >= 0) continue;
        size_t head = iperm.size();
        perm[s0] = (int32_t)iperm.size();
        iperm.push_back(s0);
        while (head < iperm.size()) {
            const int32_t v = iperm[head++];
            for (int64_t j = rp[v]; j < rp[v + 1]; ++j) {
                const int32_t w = col[j];
                if (perm[w] < 0) {
                    perm[w] = (int32_t)iperm.size();
                    iperm.push_back(w);
                }
            }
        }
    }
    for (int32_t v = 0; v < n; ++v)
        if (perm[v] < 0) {
            perm[v] = (int32_t)iperm.size();
            iperm.push_back(v);
        }
}

static GView view_of(const dbc_ctx *c) {
    GView g;
    g.rp = c->rp[c->cur];
    g.col = c->col[c->cur];
    g.scol = c->scol[c->cur];
    g.xinfo = c->ab.xinfo;
    g.xtag = c->ab.xtag;
    g.xnbr = c->ab.gnbr;
    return g;
}

static Scratch worker_scratch(const dbc_ctx *c) { return c->ws; }

static dbc_status reset_epochs(dbc_ctx *c) {
    const size_t nw = c->nscratch, n = (size_t)c->n;
    if (!nw) return DBC_OK;
    CK(cudaMemsetAsync(c->ws.mark, 0, sizeof(uint32_t) * nw * n, c->stream));
    CK(cudaMemsetAsync(c->ws.lowrec, 0, sizeof(unsigned long long) * nw * n, c->stream));
    CK(cudaMemsetAsync(c->ws.wepoch, 0, sizeof(uint32_t) * nw, c->stream));
    c->epoch_used = 0;
    return DBC_OK;
}

extern "C" dbc_status dbc_create(dbc_ctx **out, int32_t n, const int64_t *row_ptr,
                                 const int32_t *col, const int32_t *roots, int32_t k,
                                 const dbc_options *opt_in) {
    dbc_ctx *c = nullptr;
    if (!out) return fail(nullptr, DBC_EINVAL, "out is NULL");
    *out = nullptr;
    if (n < 1) return fail(nullptr, DBC_EINVAL, "n must be >= 1");
    if (!row_ptr || (!col && row_ptr && row_ptr[n] > 0)) return fail(nullptr, DBC_EINVAL, "NULL CSR");
    if (k < 0 || (k > 0 && !roots)) return fail(nullptr, DBC_EINVAL, "bad roots");
    dbc_options opt;
    if (opt_in)
        opt = *opt_in;
    else
        dbc_options_default(&opt);
    if (opt.world < 1 || opt.rank < 0 || opt.rank >= opt.world)
        return fail(nullptr, DBC_EINVAL, "bad rank/world %d/%d", opt.rank, opt.world);
    if (opt.edge_capacity < 0 || opt.workers < 0) return fail(nullptr, DBC_EINVAL, "bad sizes");
    for (int i = 0; i < 4; ++i)
        if (opt.reserved[i]) return fail(nullptr, DBC_EINVAL, "reserved fields must be zero");
    if (opt.pad0) return fail(nullptr, DBC_EINVAL, "reserved fields must be zero");
    if ((opt.dev_alloc == nullptr) != (opt.dev_free == nullptr))
        return fail(nullptr, DBC_EINVAL, "dev_alloc and dev_free come together");
    if (opt.tuning)
        for (size_t i = 0; i < sizeof(opt.tuning->reserved) / sizeof(opt.tuning->reserved[0]); ++i)
            if (opt.tuning->reserved[i]) return fail(nullptr, DBC_EINVAL, "tuning reserved fields must be zero");
    if ((opt.flags & DBC_FLAG_PULL_DELTA) && (opt.flags & DBC_FLAG_EDGE_PARALLEL))
        return fail(nullptr, DBC_EINVAL, "DBC_FLAG_PULL_DELTA excludes DBC_FLAG_EDGE_PARALLEL");
    std::vector<int32_t> h_scol;  // the rows sorted (kept for host-side batch validation)
    {
        std::string why;
        if (!validate_csr(n, row_ptr, col, why, &h_scol))
            return fail(nullptr, DBC_EINVAL, "bad CSR: %s", why.c_str());
    }
    {
        std::vector<int32_t> r(roots, roots + k);
        for (int32_t x : r)
            if (x < 0 || x >= n) return fail(nullptr, DBC_EINVAL, "root %d out of range", x);
        std::sort(r.begin(), r.end());
        if (std::adjacent_find(r.begin(), r.end()) != r.end())
            return fail(nullptr, DBC_EINVAL, "roots not distinct");
    }

    c = new dbc_ctx();
    c->dev_alloc = opt.dev_alloc;
    c->dev_free = opt.dev_free;
    c->alloc_user = opt.alloc_user;
    c->reduce = opt.reduce;
    c->reduce_user = opt.reduce_user;
    if (opt.tuning)
        c->tune = *opt.tuning;
    else
        dbc_tuning_default(&c->tune);
    const dbc_tuning &T = c->tune;
    c->device = opt.device;
    c->rank = opt.rank;
    c->world = opt.world;
    c->flags = opt.flags;
    c->n = n;
    c->k = k;
    c->nnz = c->nnz0 = row_ptr[n];
    c->h_rp.assign(row_ptr, row_ptr + (size_t)n + 1);
    c->h_scol = std::move(h_scol);
    const int64_t m = c->nnz0 / 2;
    c->edge_cap = opt.edge_capacity ? opt.edge_capacity : std::max<int64_t>(1 << 16, m / 4);
    c->col_cap = c->nnz0 + 2 * c->edge_cap;
    if (c->col_cap >= (int64_t)INT32_MAX - 1) {
        dbc_status s = fail(nullptr, DBC_EINVAL, "graph + capacity too large for int32 offsets (%lld)",
                            (long long)c->col_cap);
        delete c;
        return s;
    }
    if (opt.flags & DBC_FLAG_NO_REORDER) {
        c->perm.resize(n);
        for (int32_t v = 0; v < n; ++v) c->perm[v] = v;
        c->iperm = c->perm;
    } else {
        bfs_order(n, row_ptr, col, c->perm, c->iperm);
    }
    for (int32_t slot = opt.rank; slot < k; slot += opt.world) c->roots_local.push_back(c->perm[roots[slot]]);
    c->k_loc = (int32_t)c->roots_local.size();

    auto bail = [&](dbc_status s) {
        g_create_msg = c->msg;
        dbc_destroy(c);
        return s;
    };
    if (cudaSetDevice(c->device) != cudaSuccess) {
        cudaGetLastError();
        fail(c, DBC_ECUDA, "cudaSetDevice(%d) failed", c->device);
        return bail(DBC_ECUDA);
    }
    cudaDeviceGetAttribute(&c->nsm, cudaDevAttrMultiProcessorCount, c->device);
    if (opt.stream) {
        c->stream = (cudaStream_t)opt.stream;
    } else {
        if (cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking) != cudaSuccess) {
            fail(c, DBC_ECUDA, "stream creation failed");
            return bail(DBC_ECUDA);
        }
        c->own_stream = true;
    }
    for (auto &e : c->ev)
        if (cudaEventCreate(&e) != cudaSuccess) {
            fail(c, DBC_ECUDA, "event creation failed");
            return bail(DBC_ECUDA);
        }
    c->ev_ok = true;
    {
        int lo = 0, hi = 0;
        cudaDeviceGetStreamPriorityRange(&lo, &hi);
        if (cudaStreamCreateWithPriority(&c->hstream, cudaStreamNonBlocking, hi) != cudaSuccess ||
            cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&c->ev_prof, cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming) != cudaSuccess) {
            fail(c, DBC_ECUDA, "heavy-lane stream creation failed");
            return bail(DBC_ECUDA);
        }
    }

    // workers: persistent CTAs; bounded by roots and by a scratch-memory budget.
    // Per worker: the n-sized arrays of Scratch (mark, lowrec, dacc, Dv, Dold,
    // Dsig, U0, U1, Rv, Rl, Bq) and of the help board (gU), Doff, the deferred
    // long rows X, the insertion window (Wul, Wlev) and the chunk mirror.
    const int wcap = T.window > 0 ? T.window : kWindow;
    const size_t per_worker = (size_t)n * (4 + 8 + 8 + 4 + 4 + 8 + 4 + 4 + 4 + 4 + 4 + 4) + (size_t)(n + 2) * 4 +
                              (size_t)kXcap * sizeof(XRow) + (size_t)2 * wcap * sizeof(int32_t) +
                              sizeof(ChunkSmem) + 64;
    size_t free_b = 0, total_b = 0;
    cudaMemGetInfo(&free_b, &total_b);
    const size_t state_b = (size_t)c->k_loc * n * 24 + (size_t)c->col_cap * 8 + (size_t)n * 40;
    size_t budget = free_b > state_b ? (free_b - state_b) / 2 : 0;
    int64_t maxdeg = 0;
    for (int32_t v = 0; v < n; ++v) maxdeg = std::max<int64_t>(maxdeg, row_ptr[v + 1] - row_ptr[v]);
    // static kernel: one 1024-thread CTA per SM (64 registers) -- measured on
    // B200 against 256 (2/SM), 512 and 128 (4/SM): R-MAT 16 5.8 vs 9.6 ms,
    // Delaunay 2^18 22.3 vs 29.4 ms, Kronecker 20 0.85 vs 1.56 s
    c->sblock = 1024;
    if (T.static_block > 0) {
        const int b = T.static_block;
        c->sblock = (b == 128 || b == 512 || b == 1024) ? b : 256;
    }
    c->lowdeg = maxdeg <= 32;  // every row walked by one lane: no chunked up levels
    c->maxdeg0 = maxdeg;
    if (T.help_down_min >= 0) c->hd_min = std::max(1, T.help_down_min);
    if (T.help_down_block >= 0) c->hd_block = std::max(32, T.help_down_block);
    if (T.help_entries >= 0) c->he_entries = std::max(256, T.help_entries);
    if (T.help_min_blocks >= 0) c->he_min = std::max(1, T.help_min_blocks);
    if (T.busy_help >= 0) c->busy_help = T.busy_help;
    if (T.busy_min >= 0) c->busy_min = std::max(1, T.busy_min);
    if (T.down_long_min >= 0) c->dl_min = std::max(1, T.down_long_min);
    if (T.wide_inlane >= 0) c->wide_inlane = T.wide_inlane;
    // Update CTAs (measured on B200): one 1024-thread CTA per
    // SM (64 registers) by default -- a window-merged job has wide levels and
    // hub rows (R-MAT 16 +7.5%, Kronecker 20 +6%, small world +6% over one
    // 512-thread CTA); low-degree graphs with many roots per SM (>= 3 x #SMs,
    // long chains of narrow levels: Delaunay 2^18) run two register-capped
    // 512-thread CTAs per SM instead (+40% over 1024).
    const bool many_narrow = c->lowdeg && c->k_loc >= 3 * c->nsm;
    c->block = many_narrow ? 512 : 1024;
    if (T.update_block > 0) {
        const int b = T.update_block;
        c->block = b == 128 ? 128 : (b == 256 ? 256 : (b == 1024 ? 1024 : 512));
    }
    c->ub2 = c->block == 512 && c->k_loc >= 3 * c->nsm;
    if (T.update_pair >= 0) c->ub2 = c->block == 512 && T.update_pair != 0;
    int upb = c->block == 128 ? 4 : (c->block >= 512 ? (c->ub2 ? 2 : 1) : 2);  // update CTAs per SM
    int want = opt.workers ? opt.workers : upb * c->nsm;
    want = std::min(want, c->k_loc);
    int fit = (int)std::min<size_t>(budget / per_worker, 1 << 20);
    c->workers = std::max(0, std::min(want, fit));
    // in-lane short rows on wide up levels: lower latency, less even work --
    // worth it while the batch time is the slowest root chain (few roots per
    // worker: R-MAT 16 +8%), not when every worker has many roots (Kronecker 20)
    if (c->wide_inlane < 0) c->wide_inlane = c->k_loc <= 2 * std::max(c->workers, 1) ? 64 : 16;
    const int spb = c->sblock == 128 ? 4 : (c->sblock == 256 ? 2 : 1);  // static CTAs per SM
    c->sworkers = std::max(0, std::min({opt.workers ? opt.workers : spb * c->nsm,
                                        c->k_loc, fit}));
    c->hblock = c->block == 128 ? 256 : (c->block == 256 ? 512 : 1024);
    // only hub-heavy graphs (256-thread build) have step-bound slow roots
    // heavy lanes: the slowest root chains of the previous batch on 2x-wide CTAs
    // (hub-heavy graphs with fewer roots than worker slots: the batch time is the
    // slowest chain); 512-thread builds use 1024-thread heavy CTAs
    c->heavy_cap = (c->block == 128 || c->block == 1024 || c->ub2 || opt.workers) ? 0
                   : std::max(0, std::min(c->block == 512 ? c->nsm / 8 : c->nsm / 4, (int)(fit - c->workers)));
    if (T.heavy_cap >= 0 && c->block != 1024) c->heavy_cap = std::max(0, std::min(T.heavy_cap, (int)(fit - c->workers)));
    if (T.disable & DBC_TUNE_NO_HEAVY) c->heavy_cap = 0;
    if (c->k_loc > 0 && c->workers == 0) {
        fail(c, DBC_ENOMEM, "not enough device memory for one worker (%zu bytes)", per_worker);
        return bail(DBC_ENOMEM);
    }

    dbc_status s;
#define AL(p, cnt)                        \
    if ((s = dalloc(c, &(p), (cnt))) != DBC_OK) return bail(s);
    AL(c->rp[0], (size_t)n + 1);
    AL(c->rp[1], (size_t)n + 1);
    AL(c->col[0], (size_t)c->col_cap);
    AL(c->col[1], (size_t)c->col_cap);
    AL(c->scol[0], (size_t)c->col_cap);
    AL(c->scol[1], (size_t)c->col_cap);
    const size_t e2 = (size_t)2 * c->edge_cap;
    AL(c->ab.slot, e2);
    AL(c->ab.xtag, e2);
    AL(c->ab.gnbr, e2);
    AL(c->ab.xinfo, (size_t)n);
    AL(c->ab.xcnt, (size_t)n);
    AL(c->ab.xoff, (size_t)n);
    AL(c->ab.deg, (size_t)n + 1);
    AL(c->ab.sums, (size_t)scan_sums_capacity(n + 1));
    AL(c->ab.bad, 1);
    AL(c->ab.tmp, 2 * e2);
    c->ab.tmp_half = (int64_t)e2;
    AL(c->bu, (size_t)c->edge_cap);
    AL(c->bv, (size_t)c->edge_cap);
    const size_t kn = (size_t)c->k_loc * n;
    AL(c->d, kn);
    AL(c->sd, kn);
    AL(c->l2mask, kn);
    AL(c->mask_ds, (size_t)std::max(c->k_loc, 1));
    AL(c->bc, (size_t)n);
    AL(c->bc_ext, (size_t)n);
    AL(c->perm_d, (size_t)n);
    AL(c->roots_d, (size_t)c->k_loc);
    // per-insertion workers (update_lean.cu): one CTA per root when memory allows
    c->lean_workers = std::max(0, std::min(c->k_loc, fit));
    if (T.lean_workers > 0) c->lean_workers = std::max(1, std::min(c->lean_workers, T.lean_workers));
    if (T.disable & DBC_TUNE_NO_LEAN) c->lean_on = false;
    if (T.lean_max_batch >= 0) c->lean_max = T.lean_max_batch;
    if (T.lean_short >= 0) c->lean_short = T.lean_short;
    // per-insertion CTA width (measured on B200): hub-heavy
    // graphs need wide CTAs for their heavy levels (R-MAT 16: 512; Kronecker 20,
    // 10^6 vertices, whose heaviest jobs set a single-edge launch: 1024, 2.13 ->
    // 1.78 ms, Mode S and one job per insertion unchanged), meshes are
    // latency-bound on narrow levels (Delaunay 2^18: 256)
    c->lean_block = c->lowdeg ? 256 : (c->n >= (1 << 20) ? 1024 : 512);
    if (T.lean_block > 0) {
        const int b = T.lean_block;
        c->lean_block = (b == 256 || b == 512 || b == 1024) ? b : 128;
    }
    {  // a persistent grid: every worker resident (idle workers wait on the help board)
        const int per_sm = c->lean_block == 1024 ? lean_resident_1024()
                           : c->lean_block == 512 ? lean_resident_512()
                           : c->lean_block == 256 ? lean_resident_256() : lean_resident_128();
        c->lean_workers = std::min(c->lean_workers, std::max(1, per_sm) * c->nsm);
        // meshes (narrow levels) with more roots than resident wide workers: a
        // launch over many insertions (DBC_FLAG_NO_MERGE) runs 128-thread
        // workers so every root has one (Delaunay 2^18, 512 roots: 296 -> 512
        // workers, +50%); single-insertion launches keep the wide CTAs, whose
        // heaviest job sets the launch time
        if (c->lowdeg && T.lean_block <= 0 && c->lean_block > 128 && c->k_loc > c->lean_workers) {
            const int w = std::min({c->k_loc, fit, std::max(1, lean_resident_128()) * c->nsm});
            if (w > c->lean_workers) c->lean_narrow = w;
        }
        // hub graphs: a single-insertion launch is set by its heaviest job, which
        // wants one 128-register 512-thread CTA per SM; a launch over many
        // insertions (DBC_FLAG_NO_MERGE) wants every root resident: two
        // 64-register CTAs per SM (R-MAT 16: Mode S +9% / one job per
        // insertion +12% against a single build)
        if (T.lean_block <= 0 && c->lean_block == 512 && c->k_loc > c->lean_workers) {
            const int w = std::min({c->k_loc, fit, std::max(1, lean_resident_512x2()) * c->nsm});
            if (w > c->lean_workers) c->lean_pair = w;
        }
    }
    const size_t nwk = std::max({(size_t)c->workers + c->heavy_cap, (size_t)c->sworkers,
                                 (size_t)c->lean_workers, (size_t)c->lean_narrow,
                                 (size_t)c->lean_pair});  // both lanes; static; per-insertion
    c->nscratch = nwk;
    const size_t wn = nwk * n;
    AL(c->ws.mark, wn);
    AL(c->ws.lowrec, wn);
    AL(c->ws.dacc, wn);
    AL(c->ws.Dv, wn);
    AL(c->ws.Dold, wn);
    AL(c->ws.Dsig, wn);
    AL(c->ws.Doff, nwk * (n + 2));
    AL(c->ws.U0, wn);
    AL(c->ws.U1, wn);
    AL(c->ws.Rv, wn);
    AL(c->ws.Rl, wn);
    AL(c->ws.Bq, wn);
    AL(c->ws.X, nwk * (size_t)kXcap);
    AL(c->ws.wepoch, nwk);
    c->ws.wcap = wcap;
    AL(c->ws.Wul, nwk * (size_t)c->ws.wcap);
    AL(c->ws.Wlev, nwk * (size_t)c->ws.wcap);
    AL(c->help.word, nwk);
    AL(c->help.done, nwk);
    AL(c->help.ctx, nwk);
    AL(c->help.mir, nwk);
    AL(c->help.gapp, nwk);
    AL(c->help.gU, wn);
    AL(c->help.roots_left, 6);  // [0] live counter, [1] open wide requests, [2] idle workers, [3..5] = {k_loc, 0, 0}
    AL(c->help.low, nwk);
    AL(c->help.gbig, 2 * nwk);
    c->help.nworkers = (int)nwk;
    if (T.disable & DBC_TUNE_NO_HELP) c->help_on = false;
    AL(c->next_slot, 8);  // [0] next root, [1] heavy lane's next root / unused, [2..3] lean: roots done, idle, [4] lean: CTAs out
    if (c->lean_workers) {
        char *bd = nullptr;
        const size_t nlw = (size_t)std::max({c->lean_workers, c->lean_narrow, c->lean_pair});
        AL(bd, lean_board_bytes() * nlw);
        c->lean_board = (T.disable & DBC_TUNE_NO_LEAN_HELP) ? nullptr : (void *)bd;
        cudaMemsetAsync(bd, 0, lean_board_bytes() * nlw, c->stream);
    }
    AL(c->slots_d, (size_t)std::max(c->k_loc, 1));
    AL(c->stats, (size_t)kStAlloc);
    AL(c->err, 1);
    AL(c->root_prof, (size_t)6 * std::max(c->k_loc, 1) + 3 * nwk);  // + per-CTA {entry, loop end, exit}
    {
        const int kl[6] = {0, 0, 0, c->k_loc, 0, 0};
        if (cudaMemcpy(c->help.roots_left, kl, sizeof(kl), cudaMemcpyHostToDevice) != cudaSuccess)
            return bail(fail(c, DBC_ECUDA, "roots_left init"));
    }
    if (c->flags & DBC_FLAG_EDGE_PARALLEL) {  // Table II comparison kernel: one 512-thread CTA per SM
        c->eworkers = std::max(0, std::min<int>({c->nsm, c->k_loc, (int)nwk}));
        AL(c->esrc, (size_t)c->col_cap);
        AL(c->etag, (size_t)c->col_cap);
        AL(c->eodel, (size_t)std::max(c->eworkers, 1) * n);
    }
#undef AL

    // upload CSR (int32 offsets), roots; zero scratch
    {
        // relabelled CSR: row i = row of external vertex iperm[i], entries mapped, order kept
        std::vector<int32_t> rp32((size_t)n + 1);
        std::vector<int32_t> col2((size_t)c->nnz0);
        rp32[0] = 0;
        for (int32_t i = 0; i < n; ++i) {
            const int32_t v = c->iperm[i];
            int64_t o = rp32[i];
            for (int64_t j = row_ptr[v]; j < row_ptr[v + 1]; ++j) col2[(size_t)o++] = c->perm[col[j]];
            rp32[i + 1] = (int32_t)o;
        }
        std::vector<int32_t> srt(col2);
        {
            unsigned nt = std::max(1u, std::min(32u, std::thread::hardware_concurrency()));
            std::vector<std::thread> th;
            for (unsigned t = 0; t < nt; ++t)
                th.emplace_back([&, t] {
                    for (int64_t v = t; v < n; v += nt)
                        std::sort(srt.begin() + rp32[v], srt.begin() + rp32[v + 1]);
                });
            for (auto &x : th) x.join();
        }
        if (c->nnz0 && cudaMemcpy(c->scol[0], srt.data(), sizeof(int32_t) * c->nnz0,
                                  cudaMemcpyHostToDevice) != cudaSuccess) {
            fail(c, DBC_ECUDA, "upload failed: %s", cudaGetErrorString(cudaGetLastError()));
            return bail(DBC_ECUDA);
        }
        if (cudaMemcpy(c->rp[0], rp32.data(), sizeof(int32_t) * (n + 1), cudaMemcpyHostToDevice) != cudaSuccess ||
            (c->nnz0 && cudaMemcpy(c->col[0], col2.data(), sizeof(int32_t) * c->nnz0, cudaMemcpyHostToDevice) != cudaSuccess) ||
            cudaMemcpy(c->perm_d, c->perm.data(), sizeof(int32_t) * n, cudaMemcpyHostToDevice) != cudaSuccess ||
            (c->k_loc && cudaMemcpy(c->roots_d, c->roots_local.data(), sizeof(int32_t) * c->k_loc,
                                    cudaMemcpyHostToDevice) != cudaSuccess)) {
            fail(c, DBC_ECUDA, "upload failed: %s", cudaGetErrorString(cudaGetLastError()));
            return bail(DBC_ECUDA);
        }
    }
    if (c->workers) cudaMemsetAsync(c->ws.dacc, 0, sizeof(double) * wn, c->stream);
    if ((s = reset_epochs(c)) != DBC_OK) return bail(s);
    cudaMemsetAsync(c->bc, 0, sizeof(double) * n, c->stream);
    cudaMemsetAsync(c->err, 0, sizeof(int32_t), c->stream);
    cudaMemsetAsync(c->stats, 0, sizeof(unsigned long long) * kStAlloc, c->stream);
    if (cudaStreamSynchronize(c->stream) != cudaSuccess) {
        fail(c, DBC_ECUDA, "init failed: %s", cudaGetErrorString(cudaGetLastError()));
        return bail(DBC_ECUDA);
    }
    if (opt.nccl_id) {  // the BC all-reduce's communicator: one rank per GPU
        NcclApi &nc = nccl_api();
        if (!nc.ok) {
            fail(c, DBC_ENCCL, "NCCL unavailable: %s", nc.why.c_str());
            return bail(DBC_ENCCL);
        }
        ncclUniqueId id;
        std::memcpy(&id, opt.nccl_id, sizeof id);
        const ncclResult_t r = nc.comm_init_rank(&c->comm, c->world, id, c->rank);
        if (r != ncclSuccess) {
            c->comm = nullptr;
            fail(c, DBC_ENCCL, "ncclCommInitRank(%d of %d): %s", c->rank, c->world, nc.error_string(r));
            return bail(DBC_ENCCL);
        }
    }
    *out = c;
    return DBC_OK;
}

// fold the event times of the previous insert call into the totals (its work
// has completed whenever this is called after a stream synchronisation)
static dbc_status fold_timings(dbc_ctx *c) {
    if (c->tm_pending) {
        cudaEvent_t *e = c->ev + (c->evset ? 6 : 0);  // the previous call's set
        CK(cudaEventElapsedTime(&c->tm.append_ms, e[0], e[1]));
        CK(cudaEventElapsedTime(&c->tm.update_ms, e[2], e[3]));
        c->tm.append_ms_total += c->tm.append_ms;
        c->tm.update_ms_total += c->tm.update_ms;
        c->tm_pending = false;
    }
    if (c->tm_static) {
        CK(cudaEventElapsedTime(&c->tm.static_ms, c->ev[4], c->ev[5]));
        c->tm_static = false;
    }
    return DBC_OK;
}

// Multi-source static Brandes (msbrandes.cu) on low-diameter graphs: the
// automatic choice is mean degree >= 8 (R-MAT, Kronecker, small world; not
// meshes, whose 32 roots share no levels).
static bool use_static_ms(const dbc_ctx *c) {
    if (c->flags & DBC_FLAG_PULL_DELTA) return false;  // bitwise delta: Eq. (2) in its own order
    if (c->tune.static_ms >= 0) return c->tune.static_ms > 0;
    // low-diameter scale-free graphs: mean degree >= 8 and hubs (max degree >=
    // 16x the mean).  Measured: R-MAT 16 1.24x, Kronecker 20
    // 2.45x faster than the per-root kernel; the small world (mean 10, no hubs,
    // ~11 levels, so ~7 distinct levels per vertex among 32 roots) 2.5x slower.
    return c->n > 0 && c->nnz >= 8 * (int64_t)c->n && c->maxdeg0 * c->n >= 16 * c->nnz;
}

static StaticArgs static_args(dbc_ctx *c) {
    StaticArgs a;
    a.exact_delta = (c->flags & DBC_FLAG_PULL_DELTA) ? 1 : 0;
    a.g = view_of(c);
    a.n = c->n;
    a.k_loc = c->k_loc;
    a.roots = c->roots_d;
    a.d = c->d;
    a.sd = c->sd;
    a.l2mask = c->l2mask;
    a.mask_ds = c->mask_ds;
    a.bc = c->bc;
    a.ws = worker_scratch(c);
    a.next_slot = c->next_slot;
    a.stats = c->stats;
    a.err = c->err;
    return a;
}

// Runs the multi-source kernel over waves of 32-root groups.  *done = false
// (state untouched by the caller's view: the per-root kernel then recomputes
// everything) when a group overflowed its level lists or passed level 254,
// or when the scratch of one group does not fit.
static dbc_status static_ms(dbc_ctx *c, bool *done) {
    *done = false;
    const size_t n = (size_t)c->n;
    // roots per group: 64 (two per lane, one 64-bit mask) once there are more
    // than 32 roots, else 32
    const int R = c->tune.static_width == 32 ? 1 : c->tune.static_width == 64 ? 2 : (c->k_loc > 32 ? 2 : 1);
    const int G = 32 * R;
    const size_t mb = 4 * (size_t)R;  // bytes per mask
    const int ng_all = (c->k_loc + G - 1) / G;
    if (ng_all == 0 || n == 0) return DBC_OK;
    // row entries per task: 16 (R-MAT 16, mean degree 13), 64 from mean degree 24 (Kronecker 20)
    const int T = c->tune.static_chunk > 0 ? c->tune.static_chunk : (c->nnz >= 24 * (int64_t)n ? 64 : 16);
    const int64_t vcap = std::min<int64_t>((int64_t)n * 12, INT32_MAX / 2);
    const int64_t tcap = std::min<int64_t>(vcap + 12 * (c->nnz / T) + 1024, INT32_MAX / 2);
    const int nlev = ms_static_max_levels() + 3;
    const size_t per_group = n * (17 * G + 4 * mb) + (size_t)vcap * (4 + mb) + (size_t)tcap * 8 +
                             (size_t)nlev * 4 + ms_static_counter_bytes(1);
    int wave = std::min(ng_all, ms_static_max_groups());
    if (c->tune.static_groups > 0) {
        wave = std::min(wave, c->tune.static_groups);
    } else {
        size_t fr = 0, tot = 0;
        CK(cudaMemGetInfo(&fr, &tot));
        wave = (int)std::min<size_t>((size_t)wave, (fr / 2) / per_group);
    }
    const int grid = ms_static_resident(c->nsm, R);
    if (wave < 1 || grid < 1) return DBC_OK;
    MsArgs m;
    m.g = view_of(c);
    m.n = c->n;
    m.k_loc = c->k_loc;
    m.roots = c->roots_d;
    m.vcap = vcap;
    m.tcap = tcap;
    m.chunk = T;
    m.d = c->d;
    m.sd = c->sd;
    m.bc = c->bc;
    m.stats = c->stats;
    m.err = c->err;
    const size_t W = (size_t)wave;
    const size_t sz[] = {W * n * G * 8, W * n * G * 8, W * n * G, W * n * mb, W * n * 3 * mb, W * (size_t)vcap * 4, W * (size_t)vcap * mb,
                         W * (size_t)tcap * 8, W * (size_t)nlev * 4, ms_static_counter_bytes(wave),
                         2 * sizeof(unsigned)};
    constexpr int kBufs = sizeof(sz) / sizeof(sz[0]);
    void *buf[kBufs] = {};
    auto release = [&]() {
        for (void *p : buf) dfree(c, p);
    };
    for (int i = 0; i < kBufs; ++i)
        if (!(buf[i] = talloc(c, sz[i]))) {
            release();
            return DBC_OK;  // no room: the per-root kernel
        }
    m.sg = (double *)buf[0];
    m.q = (double *)buf[1];
    m.lv = (uint8_t *)buf[2];
    m.vis = buf[3];
    m.nm = buf[4];
    m.vq = (int32_t *)buf[5];
    m.vm = buf[6];
    m.tq = (int2 *)buf[7];
    m.toff = (int32_t *)buf[8];
    m.ctr = (int32_t *)buf[9];
    m.bar = (unsigned *)buf[10];
    std::vector<int32_t> ctr((size_t)4 * wave);
    bool ok = true;
    cudaError_t e = cudaSuccess;
    // the timed region starts after the scratch allocation (the per-root
    // kernel's scratch is allocated at dbc_create)
    if (c->flags & DBC_FLAG_TIMING) e = cudaEventRecord(c->ev[4], c->stream);
    if (e == cudaSuccess) e = cudaMemsetAsync(c->bc, 0, sizeof(double) * c->n, c->stream);
    if (e == cudaSuccess)
        e = cudaMemsetAsync(c->stats + kStStaticBytes, 0, sizeof(unsigned long long), c->stream);
    if (e == cudaSuccess)  // the kernel's phase clock (dbc_debug_counters)
        e = cudaMemsetAsync(c->stats + kStTraceN, 0, sizeof(unsigned long long), c->stream);
    for (int g0 = 0; g0 < ng_all && ok && e == cudaSuccess; g0 += wave) {
        m.g0 = g0;
        m.ng = std::min(wave, ng_all - g0);
        const size_t Gn = (size_t)m.ng;
        e = cudaMemsetAsync(m.sg, 0, Gn * n * G * 8, c->stream);
        if (e == cudaSuccess) e = cudaMemsetAsync(m.q, 0, Gn * n * G * 8, c->stream);
        if (e == cudaSuccess) e = cudaMemsetAsync(m.lv, 0xff, Gn * n * G, c->stream);
        if (e == cudaSuccess) e = cudaMemsetAsync(m.vis, 0, Gn * n * mb, c->stream);
        if (e == cudaSuccess) e = cudaMemsetAsync(m.nm, 0, Gn * n * 3 * mb, c->stream);
        if (e == cudaSuccess) e = cudaMemsetAsync(m.ctr, 0, ms_static_counter_bytes(m.ng), c->stream);
        if (e == cudaSuccess) e = cudaMemsetAsync(m.bar, 0, 2 * sizeof(unsigned), c->stream);
        if (e == cudaSuccess) e = launch_static_ms(m, R, grid, c->stream);
        if (e == cudaSuccess)
            e = cudaMemcpyAsync(ctr.data(), m.ctr, ms_static_counter_bytes(m.ng), cudaMemcpyDeviceToHost,
                                c->stream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(c->stream);
        for (int i = 0; e == cudaSuccess && i < m.ng; ++i)
            if (ctr[4 * i + 2]) ok = false;
    }
    if (e == cudaSuccess && ok) {
        launch_static_l2mask(static_args(c), c->stream);
        e = cudaGetLastError();
        // the timed region ends before the scratch is freed (cudaFree blocks the host)
        if (e == cudaSuccess && (c->flags & DBC_FLAG_TIMING)) e = cudaEventRecord(c->ev[5], c->stream);
    }
    release();
    CK(e);
    *done = ok;
    return DBC_OK;
}

extern "C" dbc_status dbc_static_compute(dbc_ctx *c) {
    if (!c) return DBC_EINVAL;
    CK(cudaSetDevice(c->device));
    const bool tm = c->flags & DBC_FLAG_TIMING;
    bool ms_done = false;
    if (c->workers && use_static_ms(c)) TRY(static_ms(c, &ms_done));  // records ev[4] itself
    if (!ms_done) {
        if (tm) CK(cudaEventRecord(c->ev[4], c->stream));
        CK(cudaMemsetAsync(c->bc, 0, sizeof(double) * c->n, c->stream));
        CK(cudaMemsetAsync(c->next_slot, 0, sizeof(int32_t), c->stream));
        c->lean_clean = false;
        CK(cudaMemsetAsync(c->stats + kStStaticBytes, 0, sizeof(unsigned long long), c->stream));
    }
    if (c->workers && !ms_done) {
        const StaticArgs a = static_args(c);
        if (c->sblock == 128)
            launch_static_128(a, c->sworkers, c->stream);
        else if (c->sblock == 512)
            launch_static_512(a, c->sworkers, c->stream);
        else if (c->sblock == 1024)
            launch_static_1024(a, c->sworkers, c->stream);
        else
            launch_static_256(a, c->sworkers, c->stream);
        CK(cudaGetLastError());
    }
    if (tm) {
        if (!ms_done) CK(cudaEventRecord(c->ev[5], c->stream));  // (static_ms records its own)
        c->tm_static = true;
    }
    c->have_state = true;
    return DBC_OK;
}

// Host-side batch validation against the host copy of the adjacency (caller
// ids): the same rules and error bits as the device validation (graph.cu):
// 1 self loop / out of range, 2 edge already present, 4 duplicate in the batch.
constexpr int64_t kHostValidateMax = 64;  // host-array batches up to this size are validated on the host
static inline uint64_t edge_key(int32_t a, int32_t b) {
    return ((uint64_t)(uint32_t)std::min(a, b) << 32) | (uint32_t)std::max(a, b);
}
static bool host_present(const dbc_ctx *c, int32_t a, int32_t b) {
    const uint64_t k = edge_key(a, b);
    if (c->h_ins.count(k)) return true;
    const int32_t lo = std::min(a, b), hi = std::max(a, b);
    return std::binary_search(c->h_scol.begin() + c->h_rp[lo], c->h_scol.begin() + c->h_rp[lo + 1], hi) &&
           !c->h_del.count(k);
}
static int host_validate(const dbc_ctx *c, const int32_t *u, const int32_t *v, int64_t cnt) {
    int bad = 0;
    std::vector<uint64_t> keys((size_t)cnt);
    for (int64_t i = 0; i < cnt; ++i) {
        const int32_t a = u[i], b = v[i];
        if (a < 0 || a >= c->n || b < 0 || b >= c->n || a == b) {
            bad |= 1;
            keys[(size_t)i] = ~0ull - (uint64_t)i;  // distinct placeholder
            continue;
        }
        if (host_present(c, a, b)) bad |= 2;
        keys[(size_t)i] = edge_key(a, b);
    }
    std::sort(keys.begin(), keys.end());
    if (std::adjacent_find(keys.begin(), keys.end()) != keys.end()) bad |= 4;
    return bad;
}
static const char *bad_batch_why(int bad) {
    return (bad & 1) ? "self loop or vertex out of range" : (bad & 2) ? "edge already present"
                                                                      : "duplicate edge within the batch";
}
// the host copy follows the device graph: inserted edges join, deleted ones leave
static void host_record_insert(dbc_ctx *c, const int32_t *u, const int32_t *v, int64_t cnt) {
    for (int64_t i = 0; i < cnt; ++i) c->h_ins.insert(edge_key(u[i], v[i]));
}
static void host_record_delete(dbc_ctx *c, const int32_t *u, const int32_t *v, int64_t cnt) {
    for (int64_t i = 0; i < cnt; ++i) {
        const uint64_t k = edge_key(u[i], v[i]);
        if (!c->h_ins.erase(k)) c->h_del.insert(k);
    }
}

static dbc_status read_stats(dbc_ctx *c, unsigned long long *h) {
    static_assert(kStAlloc > kStCount, "stats lanes");
    std::vector<unsigned long long> all(kStAlloc);
    CK(cudaMemcpyAsync(all.data(), c->stats, sizeof(unsigned long long) * kStAlloc, cudaMemcpyDeviceToHost,
                       c->stream));
    CK(cudaStreamSynchronize(c->stream));
    std::memcpy(h, all.data(), sizeof(unsigned long long) * kStCount);
    for (int l = 0; l < kStLanes; ++l)
        for (int i = 0; i < kStTraceN; ++i) h[i] += all[kStCount + (size_t)l * kStTraceN + i];
    return DBC_OK;
}

// host_validated: the batch passed host_validate (host-array calls): no device
// validation and no synchronisation -- the append and the update are enqueued
// behind whatever the stream is still running.
static dbc_status insert_device(dbc_ctx *c, const int32_t *u, const int32_t *v, int64_t cnt,
                                dbc_insert_stats *stats, bool host_validated) {
    if (!c->have_state) return fail(c, DBC_ESTATE, "dbc_static_compute must run before insertions");
    if (cnt < 0 || (cnt > 0 && (!u || !v))) return fail(c, DBC_EINVAL, "bad batch");
    if (cnt > INT32_MAX / 4) return fail(c, DBC_EINVAL, "batch too large");
    if (c->inserted + cnt > c->edge_cap)
        return fail(c, DBC_ECAPACITY, "edge capacity %lld exhausted (%lld inserted, batch %lld)",
                    (long long)c->edge_cap, (long long)c->inserted, (long long)cnt);
    if (c->scen_cap > 0 && cnt > c->scen_cap)  // before anything changes (state unchanged on error)
        return fail(c, DBC_EINVAL, "batch of %lld exceeds the scenario log (%lld insertions)",
                    (long long)cnt, (long long)c->scen_cap);
    CK(cudaSetDevice(c->device));
    const bool tm = c->flags & DBC_FLAG_TIMING;
    int launches = 0;
    // alternate event sets so the previous call's events survive until folded
    cudaEvent_t *ev = c->ev + (c->evset ? 0 : 6);
    if (tm) CK(cudaEventRecord(ev[0], c->stream));
    GView g = view_of(c);
    int32_t bad = 0;
    // the batch's per-vertex groups (and, unless validated on the host, its checks)
    launches += validate_batch(c->ab, g, c->rp[c->cur], c->n, u, v, cnt, c->nsm, c->stream, !host_validated);
    CK(cudaGetLastError());
    if (!host_validated) {
        CK(cudaMemcpyAsync(&bad, c->ab.bad, sizeof(int32_t), cudaMemcpyDeviceToHost, c->stream));
        CK(cudaStreamSynchronize(c->stream));  // all earlier work is complete here
    } else {  // DBC_FLAG_TIMING: the events fold_timings reads must be complete
        if (c->tm_pending) CK(cudaEventSynchronize((c->ev + (c->evset ? 6 : 0))[3]));
        if (c->tm_static) CK(cudaEventSynchronize(c->ev[5]));
    }
    TRY(fold_timings(c));
    // chain time per root of the previous batch (longest-first order, heavy lanes):
    // read once it is complete -- an unfinished batch leaves the older order
    if (c->prof_pending && cudaEventQuery(c->ev_prof) == cudaSuccess) {
        std::vector<unsigned long long> pr((size_t)6 * c->k_loc);
        CK(cudaMemcpy(pr.data(), c->root_prof, sizeof(unsigned long long) * pr.size(),
                      cudaMemcpyDeviceToHost));
        c->root_ms.assign(c->k_loc, 0.0);
        for (int i = 0; i < c->k_loc; ++i) c->root_ms[i] = (double)(pr[6 * i + 1] - pr[6 * i]) * 1e-6;
        c->prof_pending = false;
    }
    cudaGetLastError();  // cudaEventQuery's cudaErrorNotReady is not an error
    if (bad) return fail(c, DBC_EEDGE, "batch rejected: %s", bad_batch_why(bad));
    unsigned long long h0[kStCount] = {};
    if (stats) TRY(read_stats(c, h0));
    if (cnt == 0) {
        if (stats) std::memset(stats, 0, sizeof(*stats));
        return DBC_OK;
    }
    const int nb = 1 - c->cur;
    launches += append_batch(c->ab, c->rp[c->cur], c->col[c->cur], c->scol[c->cur], c->rp[nb],
                             c->col[nb], c->scol[nb], c->n, c->nnz, c->nsm, c->stream);
    CK(cudaGetLastError());
    c->cur = nb;
    c->nnz += 2 * cnt;
    c->inserted += cnt;
    if (tm) CK(cudaEventRecord(ev[1], c->stream));

    // epoch budget: each job of a worker consumes one epoch (30 bits available)
    const uint64_t jobs = (uint64_t)c->k_loc * (uint64_t)cnt;
    if (c->epoch_used + jobs + 1 >= (1ull << 30)) TRY(reset_epochs(c));
    c->epoch_used += jobs;

    UpdateArgs a;
    a.g = view_of(c);
    a.n = c->n;
    a.k_loc = c->k_loc;
    a.roots = c->roots_d;
    a.d = c->d;
    a.sd = c->sd;
    a.l2mask = c->l2mask;
    a.mask_ds = c->mask_ds;
    a.bc = c->bc;
    a.ins_u = u;
    a.ins_v = v;
    a.ws = worker_scratch(c);
    a.next_slot = c->next_slot;
    a.stats = c->stats;
    a.err = c->err;
    a.root_prof = c->prof_on ? c->root_prof : nullptr;
    a.slot_list = nullptr;
    a.slot_count = 0;
    a.worker_base = 0;
    a.steal_list = nullptr;
    a.steal_count = 0;
    a.steal_next = nullptr;
    a.help = HelpBoard{};  // Mode S: no cooperative help
    a.merge = (c->flags & DBC_FLAG_NO_MERGE) ? 0 : 1;
    a.scen = nullptr;
    a.del = 0;
    a.hd_min = c->hd_min;
    a.hd_block = c->hd_block;
    a.he_entries = c->he_entries;
    a.he_min = c->he_min;
    a.busy_help = c->busy_help;
    a.busy_min = c->busy_min;
    a.dl_min = c->dl_min;
    a.wide_inlane = c->wide_inlane;
    a.trace_slot = c->tune.trace_slot;
    a.lowdeg = c->lowdeg && !(c->tune.disable & DBC_TUNE_NO_LOWDEG);
    if (c->scen_cap > 0) {  // Fig. 2 / Fig. 4 log: one job per (root, insertion)
        a.scen = c->scen;
        a.merge = 0;
        c->scen_last = cnt;
    }
    if (tm) CK(cudaEventRecord(ev[2], c->stream));
    int ulaunch = 0;
    // one job per (root, insertion) -- Mode S, DBC_FLAG_NO_MERGE, the scenario
    // log, and batches too small to merge -- runs the per-insertion kernel
    const bool pull = c->flags & DBC_FLAG_PULL_DELTA;
    const bool per_ins = (c->flags & (DBC_FLAG_MODE_S | DBC_FLAG_NO_MERGE)) || a.scen || pull;
    const bool use_lean = c->lean_workers > 0 && !c->eworkers && (c->lean_on || pull) &&
                          (per_ins || cnt <= c->lean_max);
    a.static_slots = 0;
    a.lean_board = nullptr;
    a.pull_delta = pull ? 1 : 0;
    a.short_mult = c->lean_short;
    if (use_lean) {
        const bool many = !(c->flags & DBC_FLAG_MODE_S) && cnt > 1;  // one launch over many insertions
        const bool narrow = c->lean_narrow > 0 && many;
        const bool pair = c->lean_pair > 0 && many;
        const int nw = narrow ? c->lean_narrow : (pair ? c->lean_pair : c->lean_workers);
        a.lean_board = pull ? nullptr : c->lean_board;  // pull mode: every pass local
        a.merge = 0;
        a.root_prof = c->prof_on ? c->root_prof : nullptr;
        if (c->prof_on)
            CK(cudaMemsetAsync(c->root_prof, 0,
                               sizeof(unsigned long long) * (6 * std::max(c->k_loc, 1) + 3 * c->nscratch),
                               c->stream));
        const int64_t step = (c->flags & DBC_FLAG_MODE_S) ? 1 : cnt;  // Mode S: one launch per insertion
        for (int64_t i = 0; i < cnt; i += step) {
            if (!c->lean_clean)  // else the previous launch's last CTA left the counters at zero
                CK(cudaMemsetAsync(c->next_slot, 0, 5 * sizeof(int32_t), c->stream));
            c->lean_clean = true;
            a.ins_begin = (int32_t)i;
            a.ins_end = (int32_t)std::min<int64_t>(cnt, i + step);
            if (narrow)
                launch_update_lean_128(a, nw, c->stream);
            else if (pair)
                launch_update_lean_512x2(a, nw, c->stream);
            else if (c->lean_block == 1024)
                launch_update_lean_1024(a, nw, c->stream);
            else if (c->lean_block == 512)
                launch_update_lean_512(a, nw, c->stream);
            else if (c->lean_block == 256)
                launch_update_lean_256(a, nw, c->stream);
            else
                launch_update_lean_128(a, nw, c->stream);
            ++ulaunch;
        }
        CK(cudaGetLastError());
    } else if (c->eworkers) {  // edge-based parallel update (Alg. 4 / Alg. 6), one launch per insertion
        launches += launch_edge_coo(a.g, c->n, c->esrc, c->etag, c->stream);
        EdgeArgs e;
        e.g = a.g;
        e.n = c->n;
        e.k_loc = c->k_loc;
        e.roots = c->roots_d;
        e.d = c->d;
        e.sd = c->sd;
        e.bc = c->bc;
        e.ins_u = u;
        e.ins_v = v;
        e.ws = a.ws;
        e.odel = c->eodel;
        e.src = c->esrc;
        e.tag = c->etag;
        e.nnz = (int32_t)c->nnz;
        e.stats = c->stats;
        e.err = c->err;
        e.next_slot = c->next_slot;
        for (int64_t i = 0; i < cnt; ++i) {
            CK(cudaMemsetAsync(c->next_slot, 0, sizeof(int32_t), c->stream));
            c->lean_clean = false;
            e.ins = (int32_t)i;
            launch_edge_update(e, c->eworkers, c->stream);
            ++ulaunch;
        }
        CK(cudaGetLastError());
    } else if (c->workers) {
        if (!(c->flags & DBC_FLAG_MODE_S)) {
            // Mode A with heavy lanes: order slots by last chain time (longest
            // first), the slowest ones go to the wide CTAs
            a.root_prof = c->root_prof;
            const int k = c->k_loc;
            std::vector<int32_t> order(k);
            for (int i = 0; i < k; ++i) order[i] = i;
            int nh = 0;
            if ((int)c->root_ms.size() == k && k > 1) {
                std::stable_sort(order.begin(), order.end(),
                                 [&](int x, int y) { return c->root_ms[x] > c->root_ms[y]; });
                std::vector<double> srt(c->root_ms);
                std::nth_element(srt.begin(), srt.begin() + k / 2, srt.end());
                const double med = srt[k / 2];
                double hf = c->block == 512 ? 1.8 : 1.3;  // "slow" = this many medians
                if (c->tune.heavy_factor > 0.0f) hf = c->tune.heavy_factor;
                while (nh < c->heavy_cap && nh < k - 1 && c->root_ms[order[nh]] > hf * med) ++nh;
            }
            // slot list: normal slots (longest first), then the heavy ones
            std::vector<int32_t> list;
            list.reserve(k);
            for (int i = nh; i < k; ++i) list.push_back(order[i]);
            for (int i = 0; i < nh; ++i) list.push_back(order[i]);
            CK(cudaMemcpyAsync(c->slots_d, list.data(), sizeof(int32_t) * k, cudaMemcpyHostToDevice,
                               c->stream));
            CK(cudaMemsetAsync(c->next_slot, 0, 2 * sizeof(int32_t), c->stream));
            c->lean_clean = false;
            a.ins_begin = 0;
            a.ins_end = (int32_t)cnt;
            if (c->help_on) {  // fresh board: all requests closed, every root chain pending
                a.help = c->help;
                CK(cudaMemsetAsync(c->help.word, 0, sizeof(unsigned long long) * c->help.nworkers, c->stream));
                CK(cudaMemcpyAsync(c->help.roots_left, c->help.roots_left + 3, 3 * sizeof(int),
                                   cudaMemcpyDeviceToDevice, c->stream));  // no host sync per batch
            }
            if (nh > 0) {  // heavy lane first, on the high-priority stream
                CK(cudaEventRecord(c->ev_fork, c->stream));
                CK(cudaStreamWaitEvent(c->hstream, c->ev_fork, 0));
                UpdateArgs h = a;
                h.slot_list = c->slots_d + (k - nh);
                h.slot_count = nh;
                h.worker_base = c->workers;
                h.next_slot = c->next_slot + 1;
                h.steal_list = c->slots_d;  // heavy CTAs continue with normal roots
                h.steal_count = k - nh;
                h.steal_next = c->next_slot;
                if (c->hblock == 1024)
                    launch_update_1024(h, nh, c->hstream);
                else if (c->hblock == 512)
                    launch_update_512(h, nh, c->hstream);
                else
                    launch_update_256(h, nh, c->hstream);
                CK(cudaEventRecord(c->ev_join, c->hstream));
                ++ulaunch;
            }
            a.slot_list = c->slots_d;
            a.slot_count = k - nh;
            if (nh > 0) {  // normal CTAs take heavy roots the heavy lane has not started
                a.steal_list = c->slots_d + (k - nh);
                a.steal_count = nh;
                a.steal_next = c->next_slot + 1;
            }
            // Co-residency: a heavy CTA needs a whole SM, and idle workers of either
            // lane spin on the help board until every root chain is done -- so the
            // normal lane must leave the heavy lane its SMs, or a normal grid that
            // fills every SM first would wait forever for the heavy roots.
            const int upb_n = c->block == 128 ? 4 : (c->block == 256 ? 2 : (c->ub2 ? 2 : 1));
            const int wl = std::max(1, std::min(c->workers - nh * upb_n, k - nh));
            if (c->block == 128)
                launch_update_128(a, wl, c->stream);
            else if (c->block == 512)
                (c->ub2 ? launch_update_512x2 : launch_update_512)(a, wl, c->stream);
            else if (c->block == 1024)
                launch_update_1024(a, wl, c->stream);
            else
                launch_update_256(a, wl, c->stream);
            ++ulaunch;
            if (nh > 0) CK(cudaStreamWaitEvent(c->stream, c->ev_join, 0));
            CK(cudaEventRecord(c->ev_prof, c->stream));
            c->prof_pending = true;
            c->tm.heavy_roots = nh;
        } else {
            for (int64_t i = 0; i < cnt; ++i) {
                CK(cudaMemsetAsync(c->next_slot, 0, sizeof(int32_t), c->stream));
                c->lean_clean = false;
                a.ins_begin = (int32_t)i;
                a.ins_end = (int32_t)i + 1;
                if (c->block == 128)
                    launch_update_128(a, c->workers, c->stream);
                else if (c->block == 512)
                    (c->ub2 ? launch_update_512x2 : launch_update_512)(a, c->workers, c->stream);
                else if (c->block == 1024)
                    launch_update_1024(a, c->workers, c->stream);
                else
                    launch_update_256(a, c->workers, c->stream);
                ++ulaunch;
            }
        }
        CK(cudaGetLastError());
    }
    if (tm) {
        CK(cudaEventRecord(ev[3], c->stream));
        c->evset ^= 1;
        c->tm_pending = true;
    }
    launches += ulaunch;
    c->tm.update_launches = ulaunch;
    c->tm.kernel_launches = launches;
    c->tm.update_launches_total += ulaunch;
    c->tm.kernel_launches_total += launches;
    c->tm.insertions_total += cnt;
    if (stats) {
        unsigned long long h[kStCount];
        TRY(read_stats(c, h));
        stats->insertions = cnt;
        stats->case_count[0] = (int64_t)(h[kStCase1] - h0[kStCase1]);
        stats->case_count[1] = (int64_t)(h[kStCase2] - h0[kStCase2]);
        stats->case_count[2] = (int64_t)(h[kStCase3] - h0[kStCase3]);
        stats->touched = (int64_t)(h[kStTouched] - h0[kStTouched]);
        stats->down_vertices = (int64_t)(h[kStDown] - h0[kStDown]);
        stats->edges_scanned = (int64_t)(h[kStScanned] - h0[kStScanned]);
        stats->alg_bytes = (int64_t)(h[kStBytes] - h0[kStBytes]);
    }
    return DBC_OK;
}

extern "C" dbc_status dbc_insert_edges_device(dbc_ctx *c, const int32_t *u, const int32_t *v,
                                              int64_t count, dbc_insert_stats *stats) {
    if (!c) return DBC_EINVAL;
    if (count < 0 || (count > 0 && (!u || !v))) return fail(c, DBC_EINVAL, "bad batch");
    if (c->inserted + count > c->edge_cap)
        return fail(c, DBC_ECAPACITY, "edge capacity %lld exhausted (%lld inserted, batch %lld)",
                    (long long)c->edge_cap, (long long)c->inserted, (long long)count);
    if (!c->have_state) return fail(c, DBC_ESTATE, "dbc_static_compute must run before insertions");
    CK(cudaSetDevice(c->device));
    // the batch also goes to the host copy of the graph: staged in pinned memory
    // on the stream (asynchronous: no wait for earlier work here), read after
    // insert_device's synchronisation
    if (count && !c->h_pin) CK(cudaHostAlloc((void **)&c->h_pin, sizeof(int32_t) * 2 * (size_t)c->edge_cap, 0));
    if (count) {
        CK(cudaMemcpyAsync(c->h_pin, u, sizeof(int32_t) * count, cudaMemcpyDeviceToHost, c->stream));
        CK(cudaMemcpyAsync(c->h_pin + count, v, sizeof(int32_t) * count, cudaMemcpyDeviceToHost, c->stream));
    }
    map_ids(u, v, c->bu, c->bv, count, c->perm_d, c->n, c->stream);  // caller's ids -> internal
    CK(cudaGetLastError());
    const dbc_status s = insert_device(c, c->bu, c->bv, count, stats, false);  // validates, synchronises
    if (s == DBC_OK) host_record_insert(c, c->h_pin, c->h_pin + count, count);
    return s;
}

extern "C" dbc_status dbc_insert_edges(dbc_ctx *c, const int32_t *u, const int32_t *v, int64_t count,
                                       dbc_insert_stats *stats) {
    if (!c) return DBC_EINVAL;
    if (count < 0 || (count > 0 && (!u || !v))) return fail(c, DBC_EINVAL, "bad batch");
    if (c->inserted + count > c->edge_cap)
        return fail(c, DBC_ECAPACITY, "edge capacity %lld exhausted (%lld inserted, batch %lld)",
                    (long long)c->edge_cap, (long long)c->inserted, (long long)count);
    if (!c->have_state) return fail(c, DBC_ESTATE, "dbc_static_compute must run before insertions");
    if (c->scen_cap > 0 && count > c->scen_cap)  // before anything changes (state unchanged on error)
        return fail(c, DBC_EINVAL, "batch of %lld exceeds the scenario log (%lld insertions)",
                    (long long)count, (long long)c->scen_cap);
    // Small batches (single-edge and Mode-S-like calls, where a device round trip
    // dominates) are validated on the host; larger ones on the device, whose
    // validation kernels cost less than the host's lookups (R-MAT 16, batches of
    // 1,000: host validation made the end-to-end rate 4% slower).
    const bool on_host = count <= kHostValidateMax;
    if (on_host)
        if (const int bad = host_validate(c, u, v, count))  // nothing has changed yet
            return fail(c, DBC_EEDGE, "batch rejected: %s", bad_batch_why(bad));
    CK(cudaSetDevice(c->device));
    if (count) {
        CK(cudaMemcpyAsync(c->bu, u, sizeof(int32_t) * count, cudaMemcpyHostToDevice, c->stream));
        CK(cudaMemcpyAsync(c->bv, v, sizeof(int32_t) * count, cudaMemcpyHostToDevice, c->stream));
        map_ids(c->bu, c->bv, c->bu, c->bv, count, c->perm_d, c->n, c->stream);
        CK(cudaGetLastError());
    }
    const dbc_status s = insert_device(c, c->bu, c->bv, count, stats, on_host);
    if (s == DBC_OK) host_record_insert(c, u, v, count);  // (the update runs meanwhile)
    return s;
}

// Edge deletions (decremental update, R20): validated as a whole
// (host: range, self loop, duplicate pair; device: presence), then applied one
// at a time -- tombstone the edge in both rows, then one update launch over
// all local roots for that deletion (sequential semantics, as P:440 applies
// insertions).  u, v: caller ids on the HOST.
static dbc_status delete_host_ids(dbc_ctx *c, const int32_t *u, const int32_t *v, int64_t cnt,
                                  dbc_insert_stats *stats) {
    if (!c->have_state) return fail(c, DBC_ESTATE, "dbc_static_compute must run before deletions");
    if (c->flags & (DBC_FLAG_EDGE_PARALLEL | DBC_FLAG_PULL_DELTA))
        return fail(c, DBC_EINVAL, "deletions are not supported with DBC_FLAG_EDGE_PARALLEL or DBC_FLAG_PULL_DELTA");
    if (cnt > c->edge_cap) return fail(c, DBC_EINVAL, "deletion batch larger than the staging buffer");
    if (c->scen_cap > 0 && cnt > c->scen_cap)
        return fail(c, DBC_EINVAL, "batch of %lld exceeds the scenario log (%lld insertions)",
                    (long long)cnt, (long long)c->scen_cap);
    {
        std::vector<int64_t> keys((size_t)cnt);
        for (int64_t i = 0; i < cnt; ++i) {
            const int32_t a = u[i], b = v[i];
            if (a < 0 || a >= c->n || b < 0 || b >= c->n || a == b)
                return fail(c, DBC_EEDGE, "deletion batch rejected: self loop or vertex out of range");
            keys[(size_t)i] = ((int64_t)std::min(a, b) << 32) | (uint32_t)std::max(a, b);
        }
        std::sort(keys.begin(), keys.end());
        if (std::adjacent_find(keys.begin(), keys.end()) != keys.end())
            return fail(c, DBC_EEDGE, "deletion batch rejected: duplicate edge within the batch");
    }
    CK(cudaSetDevice(c->device));
    const bool tm = c->flags & DBC_FLAG_TIMING;
    cudaEvent_t *ev = c->ev + (c->evset ? 0 : 6);
    if (tm) CK(cudaEventRecord(ev[0], c->stream));
    int launches = 0;
    if (cnt) {
        CK(cudaMemcpyAsync(c->bu, u, sizeof(int32_t) * cnt, cudaMemcpyHostToDevice, c->stream));
        CK(cudaMemcpyAsync(c->bv, v, sizeof(int32_t) * cnt, cudaMemcpyHostToDevice, c->stream));
        launches += map_ids(c->bu, c->bv, c->bu, c->bv, cnt, c->perm_d, c->n, c->stream);
    }
    launches += validate_deletions(view_of(c), c->n, c->bu, c->bv, cnt, c->ab.bad, c->stream);
    CK(cudaGetLastError());
    int32_t bad = 0;
    CK(cudaMemcpyAsync(&bad, c->ab.bad, sizeof(int32_t), cudaMemcpyDeviceToHost, c->stream));
    CK(cudaStreamSynchronize(c->stream));
    TRY(fold_timings(c));
    c->prof_pending = false;  // a deletion launch is no guide to the next batch's heavy roots
    if (bad) return fail(c, DBC_EEDGE, "deletion batch rejected: edge not present");
    unsigned long long h0[kStCount] = {};
    if (stats) TRY(read_stats(c, h0));
    if (cnt == 0) {
        if (stats) std::memset(stats, 0, sizeof(*stats));
        return DBC_OK;
    }
    const uint64_t jobs = 2ull * (uint64_t)c->k_loc * (uint64_t)cnt;  // two epochs per job
    if (c->epoch_used + jobs + 1 >= (1ull << 30)) TRY(reset_epochs(c));
    c->epoch_used += jobs;
    if (tm) CK(cudaEventRecord(ev[1], c->stream));
    UpdateArgs a;
    a.g = view_of(c);
    a.n = c->n;
    a.k_loc = c->k_loc;
    a.roots = c->roots_d;
    a.d = c->d;
    a.sd = c->sd;
    a.l2mask = c->l2mask;
    a.mask_ds = c->mask_ds;
    a.bc = c->bc;
    a.ins_u = c->bu;
    a.ins_v = c->bv;
    a.ws = worker_scratch(c);
    a.next_slot = c->next_slot;
    a.stats = c->stats;
    a.err = c->err;
    a.root_prof = nullptr;
    a.slot_list = nullptr;
    a.slot_count = 0;
    a.worker_base = 0;
    a.steal_list = nullptr;
    a.steal_count = 0;
    a.steal_next = nullptr;
    a.help = HelpBoard{};
    a.merge = 0;
    a.del = 1;
    a.static_slots = 0;
    a.lean_board = nullptr;
    a.pull_delta = 0;
    a.hd_min = c->hd_min;
    a.hd_block = c->hd_block;
    a.he_entries = c->he_entries;
    a.he_min = c->he_min;
    a.busy_help = c->busy_help;
    a.busy_min = c->busy_min;
    a.dl_min = c->dl_min;
    a.wide_inlane = c->wide_inlane;
    a.trace_slot = c->tune.trace_slot;
    a.lowdeg = c->lowdeg && !(c->tune.disable & DBC_TUNE_NO_LOWDEG);
    a.scen = nullptr;
    if (c->scen_cap > 0) {
        a.scen = c->scen;
        c->scen_last = cnt;
    }
    if (tm) CK(cudaEventRecord(ev[2], c->stream));
    int ulaunch = 0;
    // One job per (root, deletion) is latency-bound like Mode S: 128-register
    // CTAs -- 512 threads, one per SM; 256 threads, two per SM, where the batch
    // runs two CTAs per SM (many roots, narrow levels: Delaunay) -- beat the
    // batch configuration (R-MAT 16 2.55k -> 2.84k deletions/s, small world
    // 3.17k -> 3.51k, Delaunay 2^18 353 -> 390/s).  An
    // explicit dbc_tuning.update_block keeps the batch configuration.
    int dblock = c->block, dworkers = c->workers;
    bool dpair = c->ub2;
    if (c->tune.update_block <= 0 && c->workers) {
        dblock = c->ub2 ? 256 : 512;
        dpair = false;
        dworkers = std::max(1, std::min({c->k_loc, (c->ub2 ? 2 : 1) * c->nsm, (int)c->nscratch}));
    }
    for (int64_t i = 0; i < cnt; ++i) {
        launches += tombstone_edge(c->rp[c->cur], c->col[c->cur], c->scol[c->cur], c->bu, c->bv, i,
                                   c->stream);
        if (c->workers) {
            CK(cudaMemsetAsync(c->next_slot, 0, sizeof(int32_t), c->stream));
            c->lean_clean = false;
            a.ins_begin = (int32_t)i;
            a.ins_end = (int32_t)i + 1;
            if (dblock == 128)
                launch_update_128(a, dworkers, c->stream);
            else if (dblock == 512)
                (dpair ? launch_update_512x2 : launch_update_512)(a, dworkers, c->stream);
            else if (dblock == 1024)
                launch_update_1024(a, dworkers, c->stream);
            else
                launch_update_256(a, dworkers, c->stream);
            ++ulaunch;
        }
    }
    CK(cudaGetLastError());
    if (tm) {
        CK(cudaEventRecord(ev[3], c->stream));
        c->evset ^= 1;
        c->tm_pending = true;
    }
    launches += ulaunch;
    c->deleted += cnt;
    host_record_delete(c, u, v, cnt);
    c->tm.update_launches = ulaunch;
    c->tm.kernel_launches = launches;
    c->tm.update_launches_total += ulaunch;
    c->tm.kernel_launches_total += launches;
    if (stats) {
        unsigned long long h[kStCount];
        TRY(read_stats(c, h));
        stats->insertions = cnt;
        stats->case_count[0] = (int64_t)(h[kStCase1] - h0[kStCase1]);
        stats->case_count[1] = (int64_t)(h[kStCase2] - h0[kStCase2]);
        stats->case_count[2] = (int64_t)(h[kStCase3] - h0[kStCase3]);
        stats->touched = (int64_t)(h[kStTouched] - h0[kStTouched]);
        stats->down_vertices = (int64_t)(h[kStDown] - h0[kStDown]);
        stats->edges_scanned = (int64_t)(h[kStScanned] - h0[kStScanned]);
        stats->alg_bytes = (int64_t)(h[kStBytes] - h0[kStBytes]);
    }
    return DBC_OK;
}

extern "C" dbc_status dbc_delete_edges(dbc_ctx *c, const int32_t *u, const int32_t *v, int64_t count,
                                       dbc_insert_stats *stats) {
    if (!c) return DBC_EINVAL;
    if (count < 0 || (count > 0 && (!u || !v))) return fail(c, DBC_EINVAL, "bad batch");
    return delete_host_ids(c, u, v, count, stats);
}

extern "C" dbc_status dbc_delete_edges_device(dbc_ctx *c, const int32_t *u, const int32_t *v,
                                              int64_t count, dbc_insert_stats *stats) {
    if (!c) return DBC_EINVAL;
    if (count < 0 || (count > 0 && (!u || !v))) return fail(c, DBC_EINVAL, "bad batch");
    CK(cudaSetDevice(c->device));
    std::vector<int32_t> hu((size_t)count), hv((size_t)count);  // the host-side batch checks
    if (count) {  // ordered after work the caller queued on the context stream
        CK(cudaMemcpyAsync(hu.data(), u, sizeof(int32_t) * count, cudaMemcpyDeviceToHost, c->stream));
        CK(cudaMemcpyAsync(hv.data(), v, sizeof(int32_t) * count, cudaMemcpyDeviceToHost, c->stream));
        CK(cudaStreamSynchronize(c->stream));
    }
    return delete_host_ids(c, hu.data(), hv.data(), count, stats);
}

static dbc_status check_err(dbc_ctx *c) {
    int32_t e = 0;
    CK(cudaMemcpyAsync(&e, c->err, sizeof e, cudaMemcpyDeviceToHost, c->stream));
    CK(cudaStreamSynchronize(c->stream));
    if (e & kErrNumeric) return fail(c, DBC_ENUMERIC, "a shortest-path count overflowed fp64");
    return DBC_OK;
}

extern "C" dbc_status dbc_synchronize(dbc_ctx *c) {
    if (!c) return DBC_EINVAL;
    CK(cudaSetDevice(c->device));
    CK(cudaStreamSynchronize(c->stream));
    return check_err(c);
}

extern "C" dbc_status dbc_get_bc_partial_device(dbc_ctx *c, double **p) {
    if (!c || !p) return DBC_EINVAL;
    CK(cudaSetDevice(c->device));
    if ((c->flags & DBC_FLAG_EXACT_BC) && c->have_state && c->k_loc)
        {
        exact_bc(c->sd, c->roots_d, c->k_loc, c->n, c->bc, c->stream);
        CK(cudaGetLastError());
    }
    gather_ext(c->bc, c->perm_d, c->n, c->bc_ext, c->stream);  // external vertex order
    CK(cudaGetLastError());
    *p = c->bc_ext;
    return DBC_OK;
}

extern "C" dbc_status dbc_get_bc_device(dbc_ctx *c, double **out) {
    if (!c || !out) return DBC_EINVAL;
    if (!c->have_state) return fail(c, DBC_ESTATE, "no state: call dbc_static_compute first");
    if (c->world > 1 && !c->comm && !c->reduce)
        return fail(c, DBC_ESTATE, "world %d: global BC needs opt.nccl_id or opt.reduce "
                                   "(or reduce dbc_get_bc_partial_device yourself)", c->world);
    double *p = nullptr;
    TRY(dbc_get_bc_partial_device(c, &p));
    // Eq. (3) over all roots: the per-rank partials summed across ranks, in
    // place on the context stream (a copy: the library keeps its own partial)
    if (c->comm) {
        NcclApi &nc = nccl_api();
        const ncclResult_t r = nc.all_reduce(p, p, (size_t)c->n, ncclFloat64, ncclSum, c->comm, c->stream);
        if (r != ncclSuccess) return fail(c, DBC_ENCCL, "ncclAllReduce: %s", nc.error_string(r));
    } else if (c->reduce && c->world > 1) {
        const int r = c->reduce(p, (int64_t)c->n, (void *)c->stream, c->reduce_user);
        if (r != 0) return fail(c, DBC_ENCCL, "reduce callback returned %d", r);
    }
    *out = p;
    return DBC_OK;
}

extern "C" dbc_status dbc_get_bc(dbc_ctx *c, double *bc) {
    if (!c || !bc) return DBC_EINVAL;
    double *p = nullptr;
    TRY(dbc_get_bc_device(c, &p));
    CK(cudaMemcpyAsync(bc, p, sizeof(double) * c->n, cudaMemcpyDeviceToHost, c->stream));
    return check_err(c);
}

extern "C" dbc_status dbc_get_root_state(dbc_ctx *c, int32_t slot, int32_t *d, double *sigma,
                                         double *delta) {
    if (!c) return DBC_EINVAL;
    if (slot < 0 || slot >= c->k || slot % c->world != c->rank)
        return fail(c, DBC_EINVAL, "slot %d not owned by rank %d", slot, c->rank);
    if (!c->have_state) return fail(c, DBC_ESTATE, "no state: call dbc_static_compute first");
    CK(cudaSetDevice(c->device));
    const size_t li = (size_t)(slot - c->rank) / c->world, n = (size_t)c->n;
    {
        std::vector<int32_t> td(n);
        std::vector<double2> ts(n);
        CK(cudaMemcpyAsync(td.data(), c->d + li * n, sizeof(int32_t) * n, cudaMemcpyDeviceToHost, c->stream));
        CK(cudaMemcpyAsync(ts.data(), c->sd + li * n, sizeof(double2) * n, cudaMemcpyDeviceToHost, c->stream));
        CK(cudaStreamSynchronize(c->stream));
        for (size_t v = 0; v < n; ++v) {
            const size_t i = (size_t)c->perm[v];
            if (d) d[v] = td[i];
            if (sigma) sigma[v] = ts[i].x;
            if (delta) delta[v] = ts[i].y;
        }
    }
    return check_err(c);
}

extern "C" dbc_status dbc_num_local_roots(const dbc_ctx *c, int32_t *k_local) {
    if (!c || !k_local) return DBC_EINVAL;
    *k_local = c->k_loc;
    return DBC_OK;
}

extern "C" dbc_status dbc_device_bytes(const dbc_ctx *c, int64_t *bytes) {
    if (!c || !bytes) return DBC_EINVAL;
    *bytes = c->bytes;
    return DBC_OK;
}

extern "C" dbc_status dbc_get_timings(dbc_ctx *c, dbc_timings *t) {
    if (!c || !t) return DBC_EINVAL;
    CK(cudaSetDevice(c->device));
    CK(cudaStreamSynchronize(c->stream));
    TRY(fold_timings(c));
    unsigned long long h[kStCount];
    TRY(read_stats(c, h));
    c->tm.static_alg_bytes = (int64_t)h[kStStaticBytes];
    c->tm.alg_bytes_total = (int64_t)(h[kStBytes] - c->bytes_base);
    *t = c->tm;
    return DBC_OK;
}

extern "C" dbc_status dbc_debug_counters(dbc_ctx *c, int64_t *out, int32_t count) {
    if (!c || !out || count < 0) return DBC_EINVAL;
    CK(cudaSetDevice(c->device));
    unsigned long long h[kStCount];
    TRY(read_stats(c, h));
    for (int i = 0; i < count && i < kStCount; ++i) out[i] = (int64_t)h[i];
    return DBC_OK;
}

extern "C" dbc_status dbc_debug_root_profile(dbc_ctx *c, int32_t enable, int64_t *out) {
    if (!c) return DBC_EINVAL;
    CK(cudaSetDevice(c->device));
    c->prof_on = enable != 0;
    if (out) {
        CK(cudaMemcpyAsync(out, c->root_prof, sizeof(int64_t) * 6 * c->k_loc, cudaMemcpyDeviceToHost,
                           c->stream));
        CK(cudaStreamSynchronize(c->stream));
    }
    return DBC_OK;
}

extern "C" dbc_status dbc_debug_cta_profile(dbc_ctx *c, int64_t *out, int64_t capacity, int64_t *count) {
    if (!c || !count) return DBC_EINVAL;
    CK(cudaSetDevice(c->device));
    *count = 3 * (int64_t)c->nscratch;
    if (out) {
        if (capacity < *count) return DBC_EINVAL;
        CK(cudaMemcpyAsync(out, c->root_prof + 6 * std::max(c->k_loc, 1), sizeof(int64_t) * *count,
                           cudaMemcpyDeviceToHost, c->stream));
        CK(cudaStreamSynchronize(c->stream));
    }
    return DBC_OK;
}

extern "C" dbc_status dbc_scenario_log(dbc_ctx *c, int64_t max_insertions) {
    if (!c || max_insertions < 0) return DBC_EINVAL;
    CK(cudaSetDevice(c->device));
    if (max_insertions > c->scen_alloc) {
        CK(cudaStreamSynchronize(c->stream));
        if (c->scen) {
            for (auto &q : c->allocs)
                if (q == (void *)c->scen) q = nullptr;
            dfree(c, c->scen);
            c->bytes -= (int64_t)(sizeof(long long) * (size_t)std::max<int64_t>(c->scen_alloc, 1) *
                                  std::max(c->k_loc, 1));
            c->scen = nullptr;
            c->scen_alloc = 0;
        }
        TRY(dalloc(c, &c->scen, (size_t)max_insertions * std::max(c->k_loc, 1)));
        c->scen_alloc = max_insertions;
    }
    c->scen_cap = max_insertions;
    c->scen_last = 0;
    return DBC_OK;
}

extern "C" dbc_status dbc_get_scenarios(dbc_ctx *c, int64_t *out, int64_t capacity, int64_t *count) {
    if (!c || !count) return DBC_EINVAL;
    CK(cudaSetDevice(c->device));
    const int64_t need = c->scen_last * c->k_loc;
    *count = need;
    if (!out) return DBC_OK;
    if (capacity < need) return fail(c, DBC_EINVAL, "scenario buffer holds %lld, need %lld",
                                     (long long)capacity, (long long)need);
    if (need > 0) {
        CK(cudaMemcpyAsync(out, c->scen, sizeof(int64_t) * need, cudaMemcpyDeviceToHost, c->stream));
        CK(cudaStreamSynchronize(c->stream));
    }
    return DBC_OK;
}

extern "C" dbc_status dbc_reset_timings(dbc_ctx *c) {
    if (!c) return DBC_EINVAL;
    CK(cudaSetDevice(c->device));
    CK(cudaStreamSynchronize(c->stream));
    TRY(fold_timings(c));
    unsigned long long h[kStCount];
    TRY(read_stats(c, h));
    c->bytes_base = h[kStBytes];
    c->tm.append_ms_total = c->tm.update_ms_total = 0.0;
    c->tm.update_launches_total = c->tm.kernel_launches_total = 0;
    c->tm.insertions_total = c->tm.alg_bytes_total = 0;
    return DBC_OK;
}
