// edge_parallel.cu -- the edge-based parallel update (Sec. III,
// Alg. 4 P:278-297 and Alg. 6), the comparison kernel family of
// Table II: node-based (update.cu) vs edge-based parallelism.
//
// One launch per insertion (the paper's structure); one CTA per
// root (persistent over the local roots).  Every level of the search is
// one or more passes of the CTA's threads over ALL visible directed edges
// (v, w) of the graph ("the edge-based approach spawns |E| threads for every
// level of the search, regardless of the amount of work"): no queues,
// the frontier is "t[v] = down and d[v] = current_depth".
//
//  down, per level L (Alg. 4):   sigma pass  -- (w, x): w down at L, d[x] = L-1:
//                                   atomicAdd(sigma[w], sigma[x])  (pull form of
//                                   line 12; exact while sigma < 2^53, larger sums
//                                   are redone in canonical order by a vertex pass
//                                   -> d/sigma bit-exact, R5)
//                                expand pass -- (w, y): w down at L: d[y] > L+1 ->
//                                   lowered (Case 3); d[y] = L+1 -> t[y] = down
//  removal (Case 3):             (w, x): w lowered from a finite level: old
//                                   predecessors x not in D lose their contribution
//  up, per level l (Alg. 6/8):   pull pass   -- (x, y): x down at l, d[y] = l+1:
//                                   atomicAdd(delta[x], sigma[x]/sigma[y]*(1+delta[y]))
//                                vertex pass -- Alg. 8: BC += delta - delta_old
//                                   (down) / Ddelta (up); delta += Ddelta (up)
//                                push pass   -- (x, p), d[p] = l-1, l >= 2: down x
//                                   pushes new - old (guard of line 10) to p
//                                   not in D; up x pushes sigma[p]/sigma[x]*Ddelta[x]
// Same arithmetic and results as the node-based kernel (d/sigma bit-exact,
// BC within rounding); only the mapping of threads to work differs.
#include "dbc_internal.cuh"

namespace dbc {
namespace {

constexpr int kEB = 512;  // threads per CTA

struct EdgeView {
    const int32_t *src, *col, *tag;  // directed entries: source, target, insertion index (-1 = base)
    int32_t nnz;
    int32_t ins;                     // this launch's batch-local insertion index (visibility bound)
    __device__ __forceinline__ bool vis(int j) const { return __ldg(tag + j) <= ins; }
};

template <class F>
__device__ __forceinline__ void for_edges(const EdgeView &e, F f) {
    for (int j = threadIdx.x; j < e.nnz; j += kEB) {
        if (!e.vis(j)) continue;
        f(j, __ldg(e.src + j), __ldg(e.col + j));
    }
}

template <class F>
__device__ __forceinline__ void for_vertices(int n, F f) {
    for (int v = threadIdx.x; v < n; v += kEB) f(v);
}

__global__ void __launch_bounds__(kEB, 1) edge_kernel(EdgeArgs a) {
    __shared__ int s_slot, s_found, s_lmax;
    const int tid = threadIdx.x;
    const int wk = blockIdx.x;
    const int n = a.n;
    uint32_t *mark = a.ws.mark + (size_t)wk * n;
    unsigned long long *lowrec = a.ws.lowrec + (size_t)wk * n;
    double *dacc = a.ws.dacc + (size_t)wk * n;
    double *osig = a.ws.Dsig + (size_t)wk * n;  // old sigma, by vertex
    double *odel = a.odel + (size_t)wk * n;     // old delta, by vertex
    uint32_t epoch = a.ws.wepoch[wk];
    EdgeView e{a.src, a.g.col, a.tag, a.nnz, a.ins};
    unsigned long long c1 = 0, c2 = 0, c3 = 0, scanned = 0, bytes = 0;

    for (;;) {
        if (tid == 0) {
            const int q = atomicAdd(a.next_slot, 1);
            s_slot = q < a.k_loc ? q : -1;
        }
        __syncthreads();
        const int slot = s_slot;
        __syncthreads();
        if (slot < 0) break;
        int32_t *d = a.d + (size_t)slot * n;
        double2 *sd = a.sd + (size_t)slot * n;
        const int s = a.roots[slot];
        const int u = __ldg(a.ins_u + a.ins), v = __ldg(a.ins_v + a.ins);
        const int du = d[u], dv = d[v];
        bytes += 8;
        if (du == dv) {  // Case 1 (both unreachable included): nothing to do
            ++c1;
            continue;
        }
        const int ul = du < dv ? v : u;
        const int L0 = min(du, dv) + 1;
        const bool case3 = max(du, dv) != L0;
        case3 ? ++c3 : ++c2;
        ++epoch;
        const uint32_t E = epoch << 2, mD = E | kDown, mU = E | kUp;
        auto oldd = [&](int w) {  // level before this insertion
            const unsigned long long r = lowrec[w];
            return ((uint32_t)(r >> 32) == epoch) ? (int)(uint32_t)r : d[w];
        };
        __syncthreads();  // every thread has read d[u], d[v]
        if (tid == 0) {
            if (case3) {
                lowrec[ul] = ((unsigned long long)epoch << 32) | (uint32_t)d[ul];
                d[ul] = L0;
            }
            mark[ul] = mD;
            osig[ul] = sd[ul].x;
            odel[ul] = sd[ul].y;
            sd[ul] = make_double2(0.0, 0.0);
            s_found = 0;
            s_lmax = L0;
        }
        __syncthreads();
        // ---------------- down phase (Alg. 4) ----------------
        int L = L0;
        for (;;) {
            // sigma of the level-L down vertices (pull)
            for_edges(e, [&](int, int w, int x) {
                if (d[w] != L || mark[w] != mD) return;
                if (d[x] == L - 1) atomicAdd(&sd[w].x, sd[x].x);
            });
            scanned += e.nnz;
            __syncthreads();
            // sums >= 2^53 depend on the order: redo them in canonical order
            for_vertices(n, [&](int w) {
                if (d[w] != L || mark[w] != mD) return;
                double sum = sd[w].x;
                if (sum >= kExact) {
                    const int2 r = row_of(a.g, w, a.ins);
                    sum = 0.0;
                    for (int j = r.x; j < r.y; ++j) {
                        const int x = ldg_i(a.g.col + j);
                        if (d[x] == L - 1) sum += sd[x].x;
                    }
                    sd[w].x = sum;
                }
                if (!(sum <= 1.7976931348623157e308)) atomicOr(a.err, kErrNumeric);
            });
            __syncthreads();
            // expand: lower (Case 3) and claim the level-L+1 down vertices
            for_edges(e, [&](int, int w, int y) {
                if (d[w] != L || mark[w] != mD) return;
                int dy = d[y];
                if (dy > L + 1) {
                    const int old = atomicMin(d + y, L + 1);
                    if (old > L + 1) lowrec[y] = ((unsigned long long)epoch << 32) | (uint32_t)old;
                    dy = L + 1;
                }
                if (dy == L + 1 && atomicMax(mark + y, mD) < E) {  // first claimer saves the old values
                    osig[y] = sd[y].x;
                    odel[y] = sd[y].y;
                    sd[y] = make_double2(0.0, 0.0);
                    s_found = 1;
                }
            });
            scanned += e.nnz;
            __syncthreads();
            const int found = s_found;
            __syncthreads();
            if (!found) break;
            if (tid == 0) s_found = 0;
            ++L;
        }
        if (tid == 0) s_lmax = L;
        __syncthreads();
        // ---------------- (0) Case-3 removal pushes ----------------
        if (case3) {
            for_edges(e, [&](int j, int w, int x) {
                if (mark[w] != mD) return;
                const int ow = oldd(w);
                if (ow == kInf || ow == d[w]) return;
                if (d[x] != ow - 1 || mark[x] == mD) return;
                if (__ldg(e.tag + j) == e.ins) return;  // the new edge carried nothing
                atomicAdd(dacc + x, -__dmul_rn(__ddiv_rn(sd[x].x, osig[w]), 1.0 + odel[w]));
                if (atomicMax(mark + x, mU) < E) atomicMax(&s_lmax, d[x]);
            });
            scanned += e.nnz;
            __syncthreads();
        }
        // ---------------- up phase (Alg. 6 + Alg. 8) ----------------
        for (int l = s_lmax; l >= 1; --l) {
            // delta of the level-l down vertices (Eq. (2) pull)
            for_edges(e, [&](int, int x, int y) {
                if (d[x] != l || mark[x] != mD || d[y] != l + 1) return;
                atomicAdd(&sd[x].y, __dmul_rn(__ddiv_rn(sd[x].x, sd[y].x), __dadd_rn(1.0, sd[y].y)));
            });
            scanned += e.nnz;
            __syncthreads();
            // Alg. 8 for level l
            for_vertices(n, [&](int x) {
                if (d[x] != l) return;
                const uint32_t m = mark[x];
                if (m == mD) {
                    if (x != s) atomicAdd(a.bc + x, sd[x].y - odel[x]);
                } else if (m == mU) {
                    const double g = dacc[x];
                    sd[x].y += g;
                    if (x != s) atomicAdd(a.bc + x, g);
                }
            });
            __syncthreads();
            if (l >= 2) {  // level-1 vertices only feed the root
                for_edges(e, [&](int j, int x, int p) {
                    if (d[x] != l || d[p] != l - 1) return;
                    const uint32_t m = mark[x];
                    if (m == mD) {
                        if (mark[p] == mD) return;
                        const double sx = sd[x].x, sp = sd[p].x;
                        double dl = __dmul_rn(__ddiv_rn(sp, sx), 1.0 + sd[x].y);
                        const int ox = oldd(x);
                        if (ox != kInf && d[p] == ox - 1 && __ldg(e.tag + j) != e.ins)
                            dl = __dsub_rn(dl, __dmul_rn(__ddiv_rn(sp, osig[x]), 1.0 + odel[x]));
                        atomicAdd(dacc + p, dl);
                        atomicMax(mark + p, mU);
                    } else if (m == mU) {
                        const double g = dacc[x];
                        if (g == 0.0) return;
                        atomicAdd(dacc + p, __dmul_rn(__ddiv_rn(sd[p].x, sd[x].x), g));
                        if (mark[p] != mD) atomicMax(mark + p, mU);
                    }
                });
                scanned += e.nnz;
            }
            __syncthreads();
        }
        // Ddelta back to all-zero (touched entries only)
        for_vertices(n, [&](int x) {
            if (mark[x] >= E && mark[x] < E + 4) dacc[x] = 0.0;
        });
        __syncthreads();
    }
    if (tid == 0) {
        a.ws.wepoch[wk] = epoch;
        atomicAdd(stat_lane(a.stats) + kStCase1, c1);
        atomicAdd(stat_lane(a.stats) + kStCase2, c2);
        atomicAdd(stat_lane(a.stats) + kStCase3, c3);
        atomicAdd(stat_lane(a.stats) + kStScanned, scanned);
        atomicAdd(stat_lane(a.stats) + kStBytes, bytes + scanned * 12ull);  // per visited entry: src, col, tag
    }
}

// directed entries -> (source, insertion index) for the edge passes
__global__ void k_edge_coo(GView g, int32_t n, int32_t *src, int32_t *tag) {
    const int v = blockIdx.x * blockDim.x + threadIdx.x;
    if (v >= n) return;
    const int rb0 = ldg_i(g.rp + v);
    const int rb = rb0 & kMask, re = ldg_i(g.rp + v + 1) & kMask;
    int nb = 0, first = 0;
    if (rb0 < 0) {
        const int2 xi = __ldg(g.xinfo + v);
        first = xi.x;
        nb = xi.y;
    }
    const int base_end = re - nb;
    for (int j = rb; j < re; ++j) {
        src[j] = v;
        tag[j] = j < base_end ? -1 : ldg_i(g.xtag + first + (j - base_end));
    }
}

}  // namespace

int launch_edge_coo(const GView &g, int32_t n, int32_t *src, int32_t *tag, cudaStream_t s) {
    k_edge_coo<<<(n + 255) / 256, 256, 0, s>>>(g, n, src, tag);
    return 1;
}

void launch_edge_update(const EdgeArgs &a, int workers, cudaStream_t s) {
    edge_kernel<<<workers, kEB, 0, s>>>(a);
}

}  // namespace dbc
