// graph_ops.h -- host-side entry points of graph.cu (batch validation, append,
// exact-BC rebase).  Internal to libdbc.  Each returns the number of kernels it
// launched (errors are picked up by the caller with cudaGetLastError).
#pragma once

#include <cstdint>

#include <cuda_runtime.h>

namespace dbc {

struct GView;

struct AppendBufs {
    int32_t *slot;   // [2*cap] arrival slot of each directed batch entry in its group
    int32_t *xtag;   // [2*cap] grouped entries: batch-local insertion index
    int32_t *gnbr;   // [2*cap] grouped entries: neighbour
    int2 *xinfo;     // [n] per flagged vertex {first grouped index, count}
    int32_t *xcnt;   // [n] batch entries per vertex
    int32_t *xoff;   // [n] group offsets (exclusive scan of xcnt)
    int32_t *deg;    // [n+1]
    int32_t *sums;   // scan block sums
    int32_t *bad;    // [1] validation result bits
    int32_t *tmp;    // [2 * tmp_half] group-sort scratch (groups of > 32 entries)
    int64_t tmp_half;  // 2 * edge capacity
};

int64_t scan_sums_capacity(int64_t n);
int validate_batch(const AppendBufs &B, const GView &g, const int32_t *rp_old, int32_t n,
                   const int32_t *u, const int32_t *v, int64_t cnt, int nsm, cudaStream_t s, bool check = true);
int validate_deletions(const GView &g, int32_t n, const int32_t *u, const int32_t *v, int64_t cnt,
                       int32_t *bad, cudaStream_t s);
int tombstone_edge(const int32_t *rp, int32_t *col, int32_t *scol, const int32_t *u, const int32_t *v,
                   int64_t i, cudaStream_t s);
int append_batch(const AppendBufs &B, const int32_t *rp_old, const int32_t *col_old,
                 const int32_t *scol_old, int32_t *rp_new, int32_t *col_new, int32_t *scol_new,
                 int32_t n, int64_t nnz_old, int nsm, cudaStream_t s);
int map_ids(const int32_t *su, const int32_t *sv, int32_t *du, int32_t *dv, int64_t cnt,
            const int32_t *perm, int32_t n, cudaStream_t s);
int gather_ext(const double *in, const int32_t *perm, int32_t n, double *out, cudaStream_t s);
int exact_bc(const double2 *sd, const int32_t *roots, int32_t k_loc, int32_t n, double *bc,
             cudaStream_t s);

}  // namespace dbc
