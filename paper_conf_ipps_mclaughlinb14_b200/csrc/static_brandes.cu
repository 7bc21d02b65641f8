// static_brandes.cu -- K1: static Brandes over the local roots (Alg. 1,
// PAPER.md P:69-124; Eqs. (2)-(3)).  Builds the per-root state that
// the dynamic update maintains, and is the GPU recompute baseline of Table III
// (the paper used Jia et al. [13] in that role).
//
// B200 design (DESIGN.md Sec. 5 K1): persistent grid, one worker CTA per root at
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

__global__ void __launch_bounds__(kBlock) static_kernel(StaticArgs a) {
    __shared__ int s_slot;
    __shared__ int s_tail;
    const int tid = threadIdx.x;
    const int w = blockIdx.x;
    const size_t n = (size_t)a.n;
    int32_t *order = a.ws.Dv + (size_t)w * n;
    int32_t *loff = a.ws.Doff + (size_t)w * (n + 2);
    unsigned long long bytes = 0;

    for (;;) {
        if (tid == 0) s_slot = atomicAdd(a.next_slot, 1);
        __syncthreads();
        const int slot = s_slot;
        __syncthreads();
        if (slot >= a.k_loc) break;
        const int s = a.roots[slot];
        int32_t *dr = a.d + (size_t)slot * n;
        double2 *sdr = a.sd + (size_t)slot * n;

        // Stage 1 (Alg. 1 lines 3-9): d = INF, sigma = delta = 0.
        for (size_t v = tid; v < n; v += kBlock) {
            dr[v] = kInf;
            sdr[v] = make_double2(0.0, 0.0);
        }
        if (tid == 0) bytes += 20ull * n;
        __syncthreads();
        if (tid == 0) {
            dr[s] = 0;
            sdr[s] = make_double2(1.0, 0.0);
            order[0] = s;
            loff[0] = 0;
            loff[1] = 1;
            s_tail = 1;
        }
        __syncthreads();

        // Stage 2: level-synchronous BFS; level L's sigma pull fused with the
        // discovery of level L+1.
        int L = 0, lb = 0, le = 1, nl = 1;
        while (lb < le) {
            const int cnt = le - lb;
            two_tier(
                cnt, a.g, INT32_MAX,
                [&](int i, int &v) { v = order[lb + i]; return true; },
                [&](int, int) { return true; },
                [&](auto Gc, int, int wv, int2 r, int gl) {
                    constexpr int G = decltype(Gc)::value;
                    double sum = 0.0;
                    unsigned long long by = 0;
                    for (int j = r.x + gl; j < r.y; j += G) {
                        const int x = ldg_i(a.g.col + j);
                        int dx = ldcg_i(dr + x);
                        by += 8;
                        if (dx == L - 1) {
                            sum += ldcg_d2(sdr + x).x;
                            by += 8;
                        } else if (dx == kInf) {
                            if (atomicCAS(dr + x, kInf, L + 1) == kInf) {
                                const int pos = atomicAdd(&s_tail, 1);
                                order[pos] = x;
                                by += 4;
                            }
                        }
                    }
                    sum = group_sum<G>(sum);
                    if constexpr (G == 32) {
                        if (sum >= kExact) {  // order-dependent rounding: canonical sum
                            if (gl == 0) {
                                sum = 0.0;
                                for (int j = r.x; j < r.y; ++j) {
                                    const int x = ldg_i(a.g.col + j);
                                    if (ldcg_i(dr + x) == L - 1) sum += ldcg_d2(sdr + x).x;
                                }
                            }
                            sum = __shfl_sync(kFull, sum, 0);
                        }
                    }
                    if (gl == 0) {
                        by += 8;
                        if (L > 0) {
                            sdr[wv].x = sum;
                            by += 8;
                            if (!(sum <= 1.7976931348623157e308)) atomicOr(a.err, kErrNumeric);
                        }
                    }
                    bytes += by;
                });
            __syncthreads();
            const int ne = s_tail;
            __syncthreads();
            lb = le;
            le = ne;
            if (tid == 0) loff[nl + 1] = le;
            ++nl;
            ++L;
        }
        __syncthreads();
        // levels 0 .. nl-2 are non-empty; loff[j] .. loff[j+1] is level j.

        // Stage 3: dependency accumulation in reverse level order (Eq. (2)),
        // BC partial += delta (Eq. (3)), root excluded (delta_s(s) = 0).
        for (int lev = nl - 2; lev >= 1; --lev) {
            const int b0 = loff[lev], b1 = loff[lev + 1];
            two_tier(
                b1 - b0, a.g, INT32_MAX,
                [&](int i, int &v) { v = order[b0 + i]; return true; },
                [&](int, int) { return true; },
                [&](auto Gc, int, int v, int2 r, int gl) {
                    constexpr int G = decltype(Gc)::value;
                    const double sv = ldcg_d2(sdr + v).x;
                    double acc = 0.0;
                    unsigned long long by = 0;
                    for (int j = r.x + gl; j < r.y; j += G) {
                        const int y = ldg_i(a.g.col + j);
                        by += 8;
                        if (ldcg_i(dr + y) == lev + 1) {
                            const double2 t = ldcg_d2(sdr + y);
                            acc += __dmul_rn(__ddiv_rn(sv, t.x), __dadd_rn(1.0, t.y));
                            by += 16;
                        }
                    }
                    acc = group_sum<G>(acc);
                    if (gl == 0) {
                        sdr[v].y = acc;
                        atomicAdd(a.bc + v, acc);
                        by += 8 + 8 + 16;
                    }
                    bytes += by;
                });
            __syncthreads();
        }
    }
    if (bytes) atomicAdd(a.stats + kStStaticBytes, bytes);
}

void launch_static(const StaticArgs &a, int workers, cudaStream_t s) {
    static_kernel<<<workers, kBlock, 0, s>>>(a);
}

}  // namespace dbc
