// graph.cu -- K5: batch validation and graph append (+ the exact-BC rebase).
//
// The paper neglects the cost of updating the graph ("We
// neglect the cost of updating the graph ... techniques ... are discussed in
// [23]").  Here the append is a handful of bulk kernels per batch: the new CSR
// is the old one with each row extended by the batch's entries in insertion
// order (canonical order, R5), written into the second graph buffer;
// rows holding batch entries are flagged so the update kernel sees, for
// insertion i, exactly the edges with insertion index <= i (Sec. IV: edges are
// "reinserted into the graph one at a time").
//
// Validation (R16): range, self loop, already present, duplicate
// within the batch -- all decided before the live graph or any state changes.
#include <algorithm>

#include "dbc_internal.cuh"
#include "graph_ops.h"

namespace dbc {

static inline unsigned blocks_for(int64_t items, int threads) {
    return (unsigned)std::max<int64_t>(1, (items + threads - 1) / threads);
}

// one warp per batch edge: range / self loop / presence in the current graph
// (insertions: present -> bit 2; deletions (absent_bit = 4): absent -> bit 4)
__global__ void k_validate_edges(GView g, int32_t n, const int32_t *u, const int32_t *v,
                                 int64_t cnt, int32_t *bad, int32_t absent_bit = 0) {
    const int lane = threadIdx.x & 31;
    const int64_t e = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (e >= cnt) return;
    const int a = u[e], b = v[e];
    if (a < 0 || a >= n || b < 0 || b >= n || a == b) {
        if (lane == 0) atomicOr(bad, 1);
        return;
    }
    const int2 ra = row_of(g, a, INT32_MAX), rb = row_of(g, b, INT32_MAX);
    const bool use_a = (ra.y - ra.x) <= (rb.y - rb.x);
    const int2 r = use_a ? ra : rb;
    const int target = use_a ? b : a;
    bool found = false;
    for (int j = r.x + lane; j < r.y; j += 32) found |= (ldg_i(g.col + j) == target);
    const bool any = __any_sync(kFull, found);
    if (lane == 0) {
        if (!absent_bit && any) atomicOr(bad, 2);
        if (absent_bit && !any) atomicOr(bad, absent_bit);
    }
}

// Deletion of edge i of the batch (u[i], v[i]): one warp per endpoint row.  The
// canonical row keeps its order with the entry replaced by a tombstone -- the
// row's own vertex, inert in every kernel (a self entry never satisfies a
// predecessor / successor / lowering test) -- and the sorted row drops the
// entry (shifted left, INT32_MAX appended: still sorted, never matched).
__global__ void k_tombstone(const int32_t *rp, int32_t *col, int32_t *scol, const int32_t *u,
                            const int32_t *v, int64_t i) {
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int a = w == 0 ? u[i] : v[i], b = w == 0 ? v[i] : u[i];
    const int rb = rp[a] & kMask, re = rp[a + 1] & kMask;
    for (int j = rb + lane; j < re; j += 32)
        if (col[j] == b) col[j] = a;
    int p = -1;
    for (int j = rb + lane; j < re; j += 32)
        if (scol[j] == b) p = j;
#pragma unroll
    for (int o = 16; o; o >>= 1) p = max(p, __shfl_xor_sync(kFull, p, o));
    if (p < 0) return;
    for (int base = p; base < re - 1; base += 32) {
        const int j = base + lane;
        const int val = (j < re - 1) ? scol[j + 1] : 0;
        __syncwarp();
        if (j < re - 1) scol[j] = val;
        __syncwarp();
    }
    if (lane == 0) scol[re - 1] = INT32_MAX;
}

int validate_deletions(const GView &g, int32_t n, const int32_t *u, const int32_t *v, int64_t cnt,
                       int32_t *bad, cudaStream_t s) {
    cudaMemsetAsync(bad, 0, sizeof(int32_t), s);
    if (!cnt) return 0;
    k_validate_edges<<<blocks_for(cnt * 32, 256), 256, 0, s>>>(g, n, u, v, cnt, bad, 4);
    return 1;
}

int tombstone_edge(const int32_t *rp, int32_t *col, int32_t *scol, const int32_t *u, const int32_t *v,
                   int64_t i, cudaStream_t s) {
    k_tombstone<<<1, 64, 0, s>>>(rp, col, scol, u, v, i);
    return 1;
}

// count directed batch entries per vertex; remember each entry's arrival slot
__global__ void k_count(const int32_t *u, const int32_t *v, int64_t cnt, int32_t n, int32_t *xcnt,
                        int32_t *slot) {
    const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= cnt) return;
    const int a = u[e], b = v[e];
    if (a < 0 || a >= n || b < 0 || b >= n) return;  // rejected by k_validate_edges
    slot[2 * e] = atomicAdd(xcnt + a, 1);
    slot[2 * e + 1] = atomicAdd(xcnt + b, 1);
}

__global__ void k_degrees(const int32_t *rp_old, const int32_t *xcnt, int32_t n, int32_t *deg) {
    const int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (x > n) return;
    deg[x] = (x == n) ? 0 : ((rp_old[x + 1] & kMask) - (rp_old[x] & kMask) + xcnt[x]);
}

// ---- exclusive scan of int32 (3 kernels: block scan, scan of block sums, add) ----
constexpr int kScanBlock = 1024;

__device__ __forceinline__ int block_exclusive_scan(int x, int *warp_sums, int *total) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    int incl = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(kFull, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) warp_sums[wid] = incl;
    __syncthreads();
    if (wid == 0) {
        int s = lane < (kScanBlock / 32) ? warp_sums[lane] : 0;
        int si = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(kFull, si, o);
            if (lane >= o) si += y;
        }
        if (lane < kScanBlock / 32) warp_sums[lane] = si - s;
        if (lane == 31) *total = si;
    }
    __syncthreads();
    return warp_sums[wid] + incl - x;
}

__global__ void __launch_bounds__(kScanBlock) k_scan_block(const int32_t *in, int32_t *out, int64_t cnt,
                                                           int32_t *sums) {
    __shared__ int ws[32];
    __shared__ int tot;
    const int64_t i = (int64_t)blockIdx.x * kScanBlock + threadIdx.x;
    const int x = i < cnt ? in[i] : 0;
    const int ex = block_exclusive_scan(x, ws, &tot);
    if (i < cnt) out[i] = ex;
    if (threadIdx.x == 0) sums[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(kScanBlock) k_scan_sums(int32_t *sums, int32_t nb) {
    __shared__ int ws[32];
    __shared__ int tot;
    int carry = 0;
    for (int base = 0; base < nb; base += kScanBlock) {
        const int i = base + threadIdx.x;
        const int x = i < nb ? sums[i] : 0;
        const int ex = block_exclusive_scan(x, ws, &tot);
        if (i < nb) sums[i] = ex + carry;
        carry += tot;
        __syncthreads();
    }
}

__global__ void k_scan_add(int32_t *out, int64_t cnt, const int32_t *sums) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < cnt) out[i] += sums[i / kScanBlock];
}

// scatter batch entries into per-vertex groups (arrival order)
__global__ void k_group_scatter(const int32_t *u, const int32_t *v, int64_t cnt, int32_t n,
                                const int32_t *xoff, const int32_t *slot, int32_t *gtag,
                                int32_t *gnbr) {
    const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= cnt) return;
    const int a = u[e], b = v[e];
    if (a < 0 || a >= n || b < 0 || b >= n) return;
    int p = xoff[a] + slot[2 * e];
    gtag[p] = (int)e;
    gnbr[p] = b;
    p = xoff[b] + slot[2 * e + 1];
    gtag[p] = (int)e;
    gnbr[p] = a;
}

// warp per vertex with batch entries: order its group by insertion index
// (canonical order), detect duplicate edges within the batch, publish xinfo.
// Groups of up to 32 entries (all but the rarest hubs) are ranked in registers,
// one entry per lane (ties broken by lane: a self loop's two entries -- the
// batch is rejected anyway -- still land in distinct slots); larger groups are
// ranked warp-cooperatively through scratch (B.tmp).
__global__ void k_group_sort(const int32_t *xcnt, const int32_t *xoff, int32_t n, int32_t *gtag,
                             int32_t *gnbr, int2 *xinfo, int32_t *bad, int32_t *sort_tmp, int64_t tmp_half) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t x = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; x < n; x += warps) {
        const int c = xcnt[x];
        if (c == 0) continue;
        const int b = xoff[x];
        if (c <= 32) {
            const int t = lane < c ? gtag[b + lane] : INT32_MAX, nb = lane < c ? gnbr[b + lane] : -1;
            int rank = 0;
            bool dup = false;
            for (int j = 0; j < c; ++j) {
                const int tj = __shfl_sync(kFull, t, j), nj = __shfl_sync(kFull, nb, j);
                rank += (tj < t) || (tj == t && j < lane);
                dup |= (j != lane) && (nj == nb);
            }
            __syncwarp();
            if (lane < c) {
                gtag[b + rank] = t;
                gnbr[b + rank] = nb;
                if (dup) atomicOr(bad, 4);
            }
        } else {
            // larger groups (hubs): each lane ranks entries k = lane, lane + 32, ...
            // against the whole group (O(c^2 / 32), duplicates found in the same
            // pass), into the group's slice of xcnt-sized scratch, then copies back
            int32_t *rt = gtag + b, *rn = gnbr + b;
            int32_t *ot = sort_tmp + b, *on = sort_tmp + tmp_half + b;
            for (int k = lane; k < c; k += 32) {
                const int t = rt[k], nb = rn[k];
                int rank = 0;
                bool dup = false;
                for (int j = 0; j < c; ++j) {
                    const int tj = rt[j];
                    rank += (tj < t) || (tj == t && j < k);
                    dup |= (j != k) && (rn[j] == nb);
                }
                ot[rank] = t;
                on[rank] = nb;
                if (dup) atomicOr(bad, 4);
            }
            __syncwarp();
            for (int k = lane; k < c; k += 32) {
                rt[k] = ot[k];
                rn[k] = on[k];
            }
        }
        if (lane == 0) xinfo[x] = make_int2(b, c);
    }
}

// Thread per old entry j (flat over all rows, so a hub row costs no more than
// its share of the entries): its row x is found by binary search of rp_old.  The
// canonical row keeps its order and moves to rp_new[x] (the batch group goes
// after it, k_place_groups); in the sorted row the entry moves right by the
// number of the group's neighbours smaller than it.
__global__ void k_copy_entries(const int32_t *__restrict__ rp_old, const int32_t *__restrict__ col_old,
                               const int32_t *__restrict__ scol_old, const int32_t *__restrict__ rp_new,
                               int32_t *__restrict__ col_new, int32_t *__restrict__ scol_new,
                               const int32_t *__restrict__ xcnt, const int32_t *__restrict__ xoff,
                               const int32_t *__restrict__ gnbr, int32_t n, int64_t nnz_old) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nnz_old; j += stride) {
        int lo = 0, hi = n;  // rp_old[lo] <= j < rp_old[hi]: the row of j is the last such lo
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if ((__ldg(rp_old + mid) & kMask) <= j) lo = mid; else hi = mid;
        }
        const int x = lo;
        const int64_t off = j - (__ldg(rp_old + x) & kMask), nb = __ldg(rp_new + x);
        col_new[nb + off] = __ldg(col_old + j);
        const int val = __ldg(scol_old + j), c = __ldg(xcnt + x);
        int less = 0;
        if (c) {
            const int g0 = __ldg(xoff + x);
            for (int k = 0; k < c; ++k) less += __ldg(gnbr + g0 + k) < val;
        }
        scol_new[nb + off + less] = val;
    }
}

// warp per vertex with a batch group (a hub can get hundreds of the batch's
// edges): the group appended after the canonical row (P:440 order), and each
// group neighbour placed in the sorted row (old entries below it by binary
// search, group entries below it by counting)
__global__ void k_place_groups(const int32_t *__restrict__ rp_old, const int32_t *__restrict__ scol_old,
                               const int32_t *__restrict__ rp_new, int32_t *__restrict__ col_new,
                               int32_t *__restrict__ scol_new, const int32_t *__restrict__ xcnt,
                               const int32_t *__restrict__ xoff, const int32_t *__restrict__ gnbr,
                               int32_t n) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t x = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; x < n; x += warps) {
        const int c = xcnt[x];
        if (c == 0) continue;
        const int ob = rp_old[x] & kMask, len = (rp_old[x + 1] & kMask) - ob, nb = rp_new[x], g0 = xoff[x];
        for (int k = lane; k < c; k += 32) {
            const int val = gnbr[g0 + k];
            col_new[nb + len + k] = val;
            int lo = 0, hi = len;  // old entries < val
            while (lo < hi) {
                const int mid = (lo + hi) >> 1;
                if (__ldg(scol_old + ob + mid) < val) lo = mid + 1; else hi = mid;
            }
            int less = 0;
            for (int q = 0; q < c; ++q) less += gnbr[g0 + q] < val;
            scol_new[nb + lo + less] = val;
        }
    }
}

__global__ void k_flag_rows(const int32_t *xcnt, int32_t n, int32_t *rp_new) {
    const int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (x < n && xcnt[x]) rp_new[x] |= (int32_t)0x80000000u;
}

int64_t scan_sums_capacity(int64_t n) { return (n + 1 + kScanBlock - 1) / kScanBlock + 1; }

static int scan_launch(const int32_t *in, int32_t *out, int64_t cnt, int32_t *sums, cudaStream_t s) {
    const int nb = (int)blocks_for(cnt, kScanBlock);
    k_scan_block<<<nb, kScanBlock, 0, s>>>(in, out, cnt, sums);
    k_scan_sums<<<1, kScanBlock, 0, s>>>(sums, nb);
    k_scan_add<<<blocks_for(cnt, 256), 256, 0, s>>>(out, cnt, sums);
    return 3;
}

int validate_batch(const AppendBufs &B, const GView &g, const int32_t *rp_old, int32_t n,
                   const int32_t *u, const int32_t *v, int64_t cnt, int nsm, cudaStream_t s, bool check) {
    int launches = 0;
    cudaMemsetAsync(B.bad, 0, sizeof(int32_t), s);
    cudaMemsetAsync(B.xcnt, 0, sizeof(int32_t) * (size_t)n, s);
    if (cnt) {
        if (check) {  // host-validated batches skip the presence test
            k_validate_edges<<<blocks_for(cnt * 32, 256), 256, 0, s>>>(g, n, u, v, cnt, B.bad);
            ++launches;
        }
        k_count<<<blocks_for(cnt, 256), 256, 0, s>>>(u, v, cnt, n, B.xcnt, B.slot);
        ++launches;
    }
    // xoff = exclusive scan of xcnt (group offsets)
    launches += scan_launch(B.xcnt, B.xoff, n, B.sums, s);
    if (cnt) {
        k_group_scatter<<<blocks_for(cnt, 256), 256, 0, s>>>(u, v, cnt, n, B.xoff, B.slot, B.xtag,
                                                            B.gnbr);
        k_group_sort<<<std::min<int64_t>(blocks_for((int64_t)n * 32, 256), (int64_t)nsm * 16), 256, 0, s>>>(
            B.xcnt, B.xoff, n, B.xtag, B.gnbr, B.xinfo, B.bad, B.tmp, B.tmp_half);
        launches += 2;
    }
    (void)rp_old;
    return launches;
}

int append_batch(const AppendBufs &B, const int32_t *rp_old, const int32_t *col_old,
                 const int32_t *scol_old, int32_t *rp_new, int32_t *col_new, int32_t *scol_new,
                 int32_t n, int64_t nnz_old, int nsm, cudaStream_t s) {
    int launches = 0;
    k_degrees<<<blocks_for((int64_t)n + 1, 256), 256, 0, s>>>(rp_old, B.xcnt, n, B.deg);
    launches += 1 + scan_launch(B.deg, rp_new, (int64_t)n + 1, B.sums, s);
    if (nnz_old > 0)
        k_copy_entries<<<std::min<int64_t>(blocks_for(nnz_old, 256), (int64_t)nsm * 64), 256, 0, s>>>(
            rp_old, col_old, scol_old, rp_new, col_new, scol_new, B.xcnt, B.xoff, B.gnbr, n, nnz_old);
    k_place_groups<<<std::min<int64_t>(blocks_for((int64_t)n * 32, 256), (int64_t)nsm * 16), 256, 0, s>>>(
        rp_old, scol_old, rp_new, col_new, scol_new, B.xcnt, B.xoff, B.gnbr, n);
    k_flag_rows<<<blocks_for(n, 256), 256, 0, s>>>(B.xcnt, n, rp_new);
    return launches + 2 + (nnz_old > 0);
}

// external -> internal vertex ids of a batch (out-of-range ids are passed
// through unchanged so validation still rejects them)
__global__ void k_map_ids(const int32_t *su, const int32_t *sv, int32_t *du, int32_t *dv, int64_t cnt,
                          const int32_t *perm, int32_t n) {
    const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= cnt) return;
    const int a = su[e], b = sv[e];
    du[e] = (a >= 0 && a < n) ? perm[a] : a;
    dv[e] = (b >= 0 && b < n) ? perm[b] : b;
}

int map_ids(const int32_t *su, const int32_t *sv, int32_t *du, int32_t *dv, int64_t cnt,
            const int32_t *perm, int32_t n, cudaStream_t s) {
    if (cnt == 0) return 0;
    k_map_ids<<<blocks_for(cnt, 256), 256, 0, s>>>(su, sv, du, dv, cnt, perm, n);
    return 1;
}

// out[v] = in[perm[v]]: internal -> external order
__global__ void k_gather_ext(const double *in, const int32_t *perm, int32_t n, double *out) {
    const int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (v < n) out[v] = in[perm[v]];
}

int gather_ext(const double *in, const int32_t *perm, int32_t n, double *out, cudaStream_t s) {
    k_gather_ext<<<blocks_for(n, 256), 256, 0, s>>>(in, perm, n, out);
    return 1;
}

// BC partial rebased as the column sum of delta over local slots (DBC_FLAG_EXACT_BC)
__global__ void k_exact_bc(const double2 *sd, const int32_t *roots, int32_t k_loc, int32_t n,
                           double *bc) {
    const int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (v >= n) return;
    double acc = 0.0;
    for (int li = 0; li < k_loc; ++li)
        if (roots[li] != v) acc += sd[(size_t)li * n + v].y;
    bc[v] = acc;
}

int exact_bc(const double2 *sd, const int32_t *roots, int32_t k_loc, int32_t n, double *bc,
             cudaStream_t s) {
    k_exact_bc<<<blocks_for(n, 256), 256, 0, s>>>(sd, roots, k_loc, n, bc);
    return 1;
}

}  // namespace dbc
