// static_brandes.cu -- K1: static Brandes over the local roots (Alg. 1,
// PAPER.md P:69-124; Eqs. (2)-(3)).  Builds the per-root state that
// the dynamic update maintains, and is the GPU recompute baseline of Table III
// (the paper used Jia et al. [13] in that role).
//
// B200 design (DESIGN.md Sec. 6 K1): persistent grid, one worker CTA per root at
// a time (roots fetched with an atomic counter -- the coarse-grained root
// parallelism of Fig. 3), level-synchronous BFS inside the CTA with
// the frontier kept as a level-ordered queue (Alg. 5's Q/QQ).  The
// forward pass over a level fuses the sigma pull of that level's vertices with
// the discovery of the next level (one row scan); the backward pass pulls delta
// in reverse level order (Eq. (2)) and adds it to the BC partial with one fp64
// atomicAdd per vertex.  Predecessors are found by the d test of P:238;
// no predecessor lists are stored.
#include "dbc_internal.cuh"

namespace dbc {

namespace {
__global__ void __launch_bounds__(kBlock, kMinBlocks) static_kernel(StaticArgs a) {
    __shared__ int s_slot;
    __shared__ int s_tail;
    __shared__ int s_nbig;
    __shared__ BigSmem S;
    const int tid = threadIdx.x;
    const int w = blockIdx.x;
    const size_t n = (size_t)a.n;
    int32_t *order = a.ws.Dv + (size_t)w * n;
    int32_t *loff = a.ws.Doff + (size_t)w * (n + 2);
    int32_t *Bq = a.ws.Bq + (size_t)w * n;
    const GView &g = a.g;
    unsigned long long bytes = 0;
    auto enq = [&](int idx) { Bq[atomicAdd(&s_nbig, 1)] = idx; };
    if (tid == 0) s_nbig = 0;

    for (;;) {
        if (tid == 0) s_slot = atomicAdd(a.next_slot, 1);
        __syncthreads();
        const int slot = s_slot;
        __syncthreads();
        if (slot >= a.k_loc) break;
        const int s = a.roots[slot];
        const Root st{a.d + (size_t)slot * n, a.sd + (size_t)slot * n};

        // Stage 1 (Alg. 1 lines 3-9): d = INF, sigma = delta = 0 (vector stores)
        for (size_t v = tid; v < n; v += kBlock) {
            st.d[v] = kInf;
            st.sd[v] = make_double2(0.0, 0.0);
        }
        if (tid == 0) bytes += 20ull * n;  // d, sigma, delta initialised
        __syncthreads();
        if (tid == 0) {
            st.d[s] = 0;
            st.sd[s].x = 1.0;
            order[0] = s;
            loff[0] = 0;
            loff[1] = 1;
            s_tail = 1;
        }
        __syncthreads();

        // Stage 2: level-synchronous BFS; level L's sigma pull fused with the
        // discovery of level L+1 (one scan of each row).
        int L = 0, lb = 0, le = 1, nl = 1;
        auto fwd_visit = [&](int x, int dx, double sx) -> double {
            if (dx == L - 1) {
                bytes += 8;  // sigma of a predecessor
                return sx;
            }
            if (dx == kInf && atomicCAS(st.d + x, kInf, L + 1) == kInf) {
                order[atomicAdd(&s_tail, 1)] = x;
                bytes += 4;
            }
            return 0.0;
        };
        auto fwd_finish = [&](int v, double sum) {
            bytes += 8;
            if (L > 0) {
                st.sd[v].x = sum;
                bytes += 8;
                if (!(sum <= 1.7976931348623157e308)) atomicOr(a.err, kErrNumeric);
            }
        };
        while (lb < le) {
            split_pass(
                le - lb, g, INT32_MAX, [&](int i, int &v) { v = order[lb + i]; return true; },
                [&](int, int v, int2 r) {
                    double sum = 0.0;  // canonical order
                    row_walk(g, st, nullptr, r, [&](int dx) { return dx == L - 1; },
                             [&](int x, int dx, double2 q, uint32_t) { sum += fwd_visit(x, dx, q.x); });
                    bytes += 8 + 8ull * (r.y - r.x);  // row bounds, col + d per entry
                    fwd_finish(v, sum);
                },
                enq);
            __syncthreads();
            const int nbig = s_nbig;
            for (int r0 = 0; r0 < nbig; r0 += kBig) {
                const int m = min(kBig, nbig - r0);
                big_load(S, m, [&](int t) { return Bq[r0 + t]; }, [&](int i) { return order[lb + i]; },
                         g, INT32_MAX);
                big_entries(S, g, st, [&](int dx) { return dx == L - 1; }, [&](int, int x, int dx, double2 q) {
                    bytes += 8;
                    return fwd_visit(x, dx, q.x);
                });
                if (tid < m) {
                    double sum = S.acc[tid];
                    const int v = S.v[tid];
                    if (sum >= kExact) {  // order-dependent rounding: canonical sum
                        const int2 r = row_of(g, v, INT32_MAX);
                        sum = 0.0;
                        for (int j = r.x; j < r.y; ++j) {
                            const int x = ldg_i(g.col + j);
                            if (st.dist(x) == L - 1) sum += st.sd[x].x;
                        }
                    }
                    fwd_finish(v, sum);
                }
                __syncthreads();
            }
            const int ne = s_tail;
            __syncthreads();
            if (tid == 0) {
                s_nbig = 0;
                loff[nl + 1] = ne;
            }
            __syncthreads();
            lb = le;
            le = ne;
            ++nl;
            ++L;
        }
        // levels 0 .. nl-2 are non-empty; loff[j] .. loff[j+1] is level j.

        // level-2 predecessor masks for the update kernel (roots of degree <= 32)
        {
            const int2 rs = row_of(g, s, INT32_MAX);
            const bool ok = rs.y - rs.x <= kMaskDeg;
            if (ok) build_l2masks(g, st, a.l2mask + (size_t)slot * n, rs, INT32_MAX);
            if (tid == 0) a.mask_ds[slot] = ok ? rs.y - rs.x : -1;
        }

        // Stage 3: dependency accumulation in reverse level order (Eq. (2)),
        // BC partial += delta (Eq. (3)), root excluded (delta_s(s) = 0).
        for (int lev = nl - 2; lev >= 1; --lev) {
            const int b0 = loff[lev], b1 = loff[lev + 1];
            auto bwd_visit = [&](double sv, int dy, double sy, double dly) -> double {
                if (dy != lev + 1) return 0.0;
                bytes += 16;  // sigma, delta of a successor
                return __dmul_rn(__ddiv_rn(sv, sy), __dadd_rn(1.0, dly));
            };
            auto bwd_finish = [&](int v, double acc) {
                st.sd[v].y = acc;
                atomicAdd(a.bc + v, acc);
                bytes += 8 + 8 + 16;
            };
            split_pass(
                b1 - b0, g, INT32_MAX, [&](int i, int &v) { v = order[b0 + i]; return true; },
                [&](int, int v, int2 r) {
                    const double sv = st.sd[v].x;
                    double acc = 0.0;
                    row_walk(g, st, nullptr, r, [&](int dy) { return dy == lev + 1; },
                             [&](int, int dy, double2 q, uint32_t) { acc += bwd_visit(sv, dy, q.x, q.y); });
                    bytes += 8 + 8 + 8ull * (r.y - r.x);
                    bwd_finish(v, acc);
                },
                enq);
            __syncthreads();
            const int nbig = s_nbig;
            for (int r0 = 0; r0 < nbig; r0 += kBig) {
                const int m = min(kBig, nbig - r0);
                big_load(S, m, [&](int t) { return Bq[r0 + t]; }, [&](int i) { return order[b0 + i]; },
                         g, INT32_MAX);
                if (tid < m) S.c0[tid] = st.sd[S.v[tid]].x;
                __syncthreads();
                big_entries(S, g, st, [&](int dy) { return dy == lev + 1; }, [&](int t, int, int dy, double2 q) {
                    bytes += 8;
                    return bwd_visit(S.c0[t], dy, q.x, q.y);
                });
                if (tid < m) {
                    double acc = S.acc[tid];
                    if (a.exact_delta) {  // DBC_FLAG_PULL_DELTA: Eq. (2) left to right in canonical order
                        const int v = S.v[tid];
                        const int2 r = row_of(g, v, INT32_MAX);
                        const double sv = S.c0[tid];
                        acc = 0.0;
                        for (int j = r.x; j < r.y; ++j) {
                            const int y = ldg_i(g.col + j);
                            if (st.dist(y) != lev + 1) continue;
                            const double2 q = st.sd[y];
                            acc = __dadd_rn(acc, __dmul_rn(__ddiv_rn(sv, q.x), __dadd_rn(1.0, q.y)));
                        }
                    }
                    bwd_finish(S.v[tid], acc);
                }
                __syncthreads();
            }
            __syncthreads();
            if (tid == 0) s_nbig = 0;
            __syncthreads();
        }
    }
    stat_add_warp(a.stats, kStStaticBytes, bytes);
}

}  // namespace

#define DBC_CAT2(a, b) a##b
#define DBC_CAT(a, b) DBC_CAT2(a, b)
void DBC_CAT(launch_static_, DBC_BLOCK)(const StaticArgs &a, int workers, cudaStream_t s) {
    static_kernel<<<workers, kBlock, 0, s>>>(a);
}

}  // namespace dbc
