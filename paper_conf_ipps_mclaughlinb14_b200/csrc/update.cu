// update.cu -- K2/K3/K4: the per-root incremental update after an edge
// insertion (u, v) (Sec. II-D and III; Algs. 2-8), fused in
// one persistent kernel.
//
// Per (root s, insertion i), inside one worker CTA:
//  classify (K2; "trivial"): Case 1 iff d_s(u) == d_s(v)
//      (both unreachable included) -> no work; else u_high = the closer endpoint.
//  seed   (replaces Alg. 3's O(n) init): Case 3 lowers d[u_low] to
//      d[u_high]+1 (remembering the old d, possibly INF); D = {u_low}.
//  down   (K3; Alg. 2 stage 2 P:178-197, Alg. 5): level-synchronous
//      BFS over the NEW shortest-path DAG from u_low.  Each w at level L gets
//      sigma[w] = sum of sigma[x], x in adj(w), d[x] = L-1, summed in canonical
//      adjacency order (pull form -- bit-exact with the oracle; R5);
//      neighbours y with d[y] > L+1 are pulled up with atomicMin (Case 3, the
//      first lowerer records the old d); neighbours with d[y] = L+1 are claimed
//      (epoch-tagged flag, Alg. 2's t[v] = down) and queued for level L+1.
//  up     (K4; Alg. 2 stage 3 P:198-235, Alg. 7, Alg. 8
//      fused): (0) Case-3 removal pushes: every pulled-up w gives each old
//      predecessor x not in D  Ddelta[x] -= sigma[x]/sigma_old(w)*(1+delta_old(w));
//      then for l = deepest touched level down to 1:
//        down vertex x: delta_new = sum_{y succ} sigma[x]/sigma[y]*(1+delta[y])
//          (Eq. (2) by pull), BC[x] += delta_new - delta_old, and each
//          predecessor p not in D gets Ddelta[p] += new - old contribution (old
//          only for an old predecessor, and never over the new edge: the guard
//          "v != u_high or w != u_low" of Alg. 2 line 32);
//        up vertex x (t[x] = up): delta[x] += Ddelta[x], BC[x] += Ddelta[x], and
//          if l >= 2 push sigma[p]/sigma[x]*Ddelta[x] to its predecessors.
//      sigma and delta are updated in place; flags/accumulators are reset only
//      on touched entries (no O(n) Alg. 3 / Alg. 8 sweeps).
//
// Mode A (default): a worker owns one root for the whole batch and walks the
// insertions in order -- roots are independent except for BC, so no
// cross-root barrier per insertion.  Mode S: one launch per insertion.  The
// adjacency is filtered by insertion index, so both see exactly the graph the
// sequential semantics prescribes.
#include "dbc_internal.cuh"

namespace dbc {

__device__ __forceinline__ int append_smem(int *ctr) { return atomicAdd(ctr, 1); }

__global__ void __launch_bounds__(kBlock) update_kernel(UpdateArgs a) {
    __shared__ int s_slot;
    __shared__ int s_dcnt;   // |D| (absolute positions in Dv)
    __shared__ int s_ucnt;   // next up frontier size
    __shared__ int s_rcnt;   // |R|
    __shared__ int s_rmax;   // deepest removal-push target level
    __shared__ uint32_t s_work[kWarps];  // window classification bits (1 = Case 2/3)
    __shared__ int s_job[4];             // uh, ul, L0, case3 of the current job
    const int tid = threadIdx.x;
    const int wk = blockIdx.x;
    const size_t n = (size_t)a.n;

    uint32_t *mark = a.ws.mark + (size_t)wk * n;
    unsigned long long *lowrec = a.ws.lowrec + (size_t)wk * n;
    double *dacc = a.ws.dacc + (size_t)wk * n;
    int32_t *Dv = a.ws.Dv + (size_t)wk * n;
    int32_t *Dold = a.ws.Dold + (size_t)wk * n;
    double *Dsig = a.ws.Dsig + (size_t)wk * n;
    int32_t *Doff = a.ws.Doff + (size_t)wk * (n + 2);
    int32_t *Ua = a.ws.U0 + (size_t)wk * n;
    int32_t *Ub = a.ws.U1 + (size_t)wk * n;
    int32_t *Rv = a.ws.Rv + (size_t)wk * n;
    int32_t *Rl = a.ws.Rl + (size_t)wk * n;
    uint32_t epoch = a.ws.wepoch[wk];

    unsigned long long st_bytes = 0, st_scanned = 0, st_touched = 0, st_down = 0;
    unsigned long long st_case[3] = {0, 0, 0};

    for (;;) {
        if (tid == 0) s_slot = atomicAdd(a.next_slot, 1);
        __syncthreads();
        const int slot = s_slot;
        __syncthreads();
        if (slot >= a.k_loc) break;
        (void)a.roots;
        int32_t *dr = a.d + (size_t)slot * n;
        double2 *sdr = a.sd + (size_t)slot * n;

        // Insertions are walked in order.  Classification (K2) of a window of
        // kBlock insertions runs in parallel against the current d; a Case-2
        // job leaves d unchanged so the window stays valid, a Case-3 job
        // lowers distances, so the window is re-classified after it.
        int ins = a.ins_begin;
        while (ins < a.ins_end) {
            const int wend = min(ins + kBlock, a.ins_end);
            {
                const int j = ins + tid;
                bool work = false;
                if (j < wend) {
                    const int u = __ldg(a.ins_u + j), v = __ldg(a.ins_v + j);
                    work = ldcg_i(dr + u) != ldcg_i(dr + v);
                }
                const unsigned bal = __ballot_sync(kFull, work);
                if ((tid & 31) == 0) s_work[tid >> 5] = bal;
            }
            __syncthreads();
            int p = ins;
            for (; p < wend; ++p) {
                const int off = p - ins;
                if (!((s_work[off >> 5] >> (off & 31)) & 1u)) {  // Case 1: no work
                    if (tid == 0) {
                        st_case[0]++;
                        st_bytes += 8;
                    }
                    continue;
                }
                // ---------------- classify + seed (tid 0, broadcast) ----------------
                ++epoch;
                const uint32_t E = epoch << 2;
                const uint32_t mD = E | kDown, mU = E | kUp;
                if (tid == 0) {
                    const int u = __ldg(a.ins_u + p), v = __ldg(a.ins_v + p);
                    const int du = ldcg_i(dr + u), dv = ldcg_i(dr + v);
                    const bool u_is_high = du < dv;
                    const int uh = u_is_high ? u : v, ul = u_is_high ? v : u;
                    const int dh = u_is_high ? du : dv, dlo = u_is_high ? dv : du;
                    const int L0 = dh + 1;
                    const bool c3 = dlo > L0;
                    st_case[c3 ? 2 : 1]++;
                    st_bytes += 8;
                    if (c3) {
                        lowrec[ul] = ((unsigned long long)epoch << 32) | (uint32_t)dlo;
                        dr[ul] = L0;
                    }
                    mark[ul] = mD;
                    Dv[0] = ul;
                    Doff[0] = 0;
                    Doff[1] = 1;
                    s_dcnt = 1;
                    s_ucnt = 0;
                    s_rcnt = 0;
                    s_rmax = 0;
                    s_job[0] = uh;
                    s_job[1] = ul;
                    s_job[2] = L0;
                    s_job[3] = c3;
                }
                __syncthreads();
                const int uh = s_job[0], ul = s_job[1], L0 = s_job[2];
                const bool case3 = s_job[3] != 0;
                const int lim = p;  // graph as of this insertion (edge p included)

                // ---------------- down phase (K3) ----------------
                int L = L0, lb = 0, le = 1, nlev = 1;
                while (true) {
                    two_tier(
                        le - lb, a.g, lim,
                        [&](int i, int &w) { w = Dv[lb + i]; return true; },
                        [&](int, int) { return true; },
                        [&](auto Gc, int i, int w, int2 r, int gl) {
                            constexpr int G = decltype(Gc)::value;
                            const int idx = lb + i;
                            double sum = 0.0;
                            unsigned long long by = 0, sc = 0;
                            for (int j = r.x + gl; j < r.y; j += G) {
                                const int y = ldg_i(a.g.col + j);
                                int dy = ldcg_i(dr + y);
                                ++sc;
                                if (dy == L - 1) {
                                    sum += ldcg_d2(sdr + y).x;
                                    by += 8;
                                } else if (dy > L + 1) {
                                    const int old = atomicMin(dr + y, L + 1);
                                    if (old > L + 1) {
                                        lowrec[y] = ((unsigned long long)epoch << 32) | (uint32_t)old;
                                        by += 4;
                                    }
                                    dy = L + 1;
                                }
                                if (dy == L + 1) {
                                    if (atomicMax(mark + y, mD) < mD) {
                                        Dv[append_smem(&s_dcnt)] = y;
                                    }
                                }
                            }
                            sum = group_sum<G>(sum);
                            if constexpr (G == 32) {
                                if (sum >= kExact) {  // not provably exact: canonical-order sum
                                    if (gl == 0) {
                                        sum = 0.0;
                                        for (int j = r.x; j < r.y; ++j) {
                                            const int y = ldg_i(a.g.col + j);
                                            if (ldcg_i(dr + y) == L - 1) sum += ldcg_d2(sdr + y).x;
                                        }
                                    }
                                    sum = __shfl_sync(kFull, sum, 0);
                                }
                            }
                            if (gl == 0) {
                                const unsigned long long lr = ldcg_ull(lowrec + w);
                                const int od = ((uint32_t)(lr >> 32) == epoch) ? (int)(uint32_t)lr : L;
                                Dold[idx] = od;
                                Dsig[idx] = ldcg_d2(sdr + w).x;
                                sdr[w].x = sum;
                                if (!(sum <= 1.7976931348623157e308)) atomicOr(a.err, kErrNumeric);
                                by += 8 + 8 + 20;
                            }
                            st_bytes += by + 8 * sc;
                            st_scanned += sc;
                        });
                    __syncthreads();
                    const int ne = s_dcnt;
                    __syncthreads();
                    if (ne == le) break;
                    lb = le;
                    le = ne;
                    ++nlev;
                    if (tid == 0) Doff[nlev] = le;
                    ++L;
                }
                // D levels: level L0 + j occupies Dv[Doff[j] .. Doff[j+1]), j < nlev
                const int LmaxD = L0 + nlev - 1;
                const int dtotal = le;
                if (tid == 0) {
                    st_down += dtotal;
                    st_touched += dtotal;
                }

                // ---------------- (0) Case-3 removal pushes ----------------
                if (case3) {
                    for (int j = 0; j < nlev; ++j) {
                        const int b0 = Doff[j], b1 = Doff[j + 1];
                        const int lev = L0 + j;
                        two_tier(
                            b1 - b0, a.g, lim,
                            [&](int i, int &w) {
                                const int od = Dold[b0 + i];
                                w = Dv[b0 + i];
                                return od != lev && od != kInf;
                            },
                            [&](int, int) { return true; },
                            [&](auto Gc, int i, int w, int2 r, int gl) {
                                constexpr int G = decltype(Gc)::value;
                                const int idx = b0 + i;
                                const int od = Dold[idx];
                                const double osig = Dsig[idx];
                                const double coef = 1.0 + ldcg_d2(sdr + w).y;  // delta still old
                                unsigned long long by = 0, sc = 0;
                                for (int j2 = r.x + gl; j2 < r.y; j2 += G) {
                                    const int x = ldg_i(a.g.col + j2);
                                    ++sc;
                                    if (ldcg_i(dr + x) != od - 1) continue;
                                    if (x == uh && w == ul) continue;
                                    const uint32_t mx = ldcg_u(mark + x);
                                    if (mx == mD) continue;
                                    const double sx = ldcg_d2(sdr + x).x;
                                    atomicAdd(dacc + x, -__dmul_rn(__ddiv_rn(sx, osig), coef));
                                    by += 24;
                                    if (atomicMax(mark + x, mU) < E) {
                                        const int pos = append_smem(&s_rcnt);
                                        Rv[pos] = x;
                                        Rl[pos] = od - 1;
                                        atomicMax(&s_rmax, od - 1);
                                    }
                                }
                                if (gl == 0) by += 8 + 8;
                                st_bytes += by + 8 * sc;
                                st_scanned += sc;
                            });
                    }
                    __syncthreads();
                }
                const int rcnt = s_rcnt;
                const int Lmax = max(LmaxD, s_rmax);
                if (tid == 0) st_touched += rcnt;

                // ---------------- up phase (K4 + Alg. 8) ----------------
                int *Ucur = Ua, *Unext = Ub;
                int ucnt = 0;
                for (int l = Lmax; l >= 1; --l) {
                    if (l < L0 && ucnt == 0) break;  // nothing left above the insertion
                    // down vertices at level l
                    if (l >= L0 && l <= LmaxD) {
                        const int b0 = Doff[l - L0], b1 = Doff[l - L0 + 1];
                        two_tier(
                            b1 - b0, a.g, lim,
                            [&](int i, int &x) { x = Dv[b0 + i]; return true; },
                            [&](int, int) { return true; },
                            [&](auto Gc, int i, int x, int2 r, int gl) {
                                constexpr int G = decltype(Gc)::value;
                                const int idx = b0 + i;
                                const double2 sx2 = ldcg_d2(sdr + x);
                                const double sx = sx2.x, odel = sx2.y;
                                double acc = 0.0;
                                unsigned long long by = 0, sc = 0;
                                for (int j = r.x + gl; j < r.y; j += G) {
                                    const int y = ldg_i(a.g.col + j);
                                    ++sc;
                                    if (ldcg_i(dr + y) == l + 1) {
                                        const double2 t = ldcg_d2(sdr + y);
                                        acc += __dmul_rn(__ddiv_rn(sx, t.x), __dadd_rn(1.0, t.y));
                                        by += 16;
                                    }
                                }
                                acc = group_sum<G>(acc);
                                if (l >= 2) {
                                    const bool not_pulled = Dold[idx] == l;
                                    const double osig = Dsig[idx];
                                    const double cnew = 1.0 + acc, cold = 1.0 + odel;
                                    for (int j = r.x + gl; j < r.y; j += G) {
                                        const int p = ldg_i(a.g.col + j);
                                        ++sc;
                                        if (ldcg_i(dr + p) != l - 1) continue;
                                        const uint32_t mp = ldcg_u(mark + p);
                                        if (mp == mD) continue;
                                        const double sp = ldcg_d2(sdr + p).x;
                                        double dlt = __dmul_rn(__ddiv_rn(sp, sx), cnew);
                                        if (not_pulled && !(p == uh && x == ul))
                                            dlt = __dsub_rn(dlt, __dmul_rn(__ddiv_rn(sp, osig), cold));
                                        atomicAdd(dacc + p, dlt);
                                        by += 24;
                                        if (atomicMax(mark + p, mU) < E) Unext[append_smem(&s_ucnt)] = p;
                                    }
                                }
                                group_sync<G>();
                                if (gl == 0) {
                                    sdr[x].y = acc;
                                    atomicAdd(a.bc + x, acc - odel);
                                    by += 8 + 16 + 16;
                                }
                                st_bytes += by + 8 * sc;
                                st_scanned += sc;
                            });
                    }
                    // up vertices at level l found by level l+1
                    two_tier(
                        ucnt, a.g, lim,
                        [&](int i, int &x) { x = Ucur[i]; return true; },
                        [&](int, int) { return l >= 2; },
                        [&](auto Gc, int, int x, int2 r, int gl) {
                            constexpr int G = decltype(Gc)::value;
                            const double g = ldcg_d(dacc + x);
                            unsigned long long by = 0, sc = 0;
                            if (g != 0.0) {
                                const double sx = ldcg_d2(sdr + x).x;
                                for (int j = r.x + gl; j < r.y; j += G) {
                                    const int p = ldg_i(a.g.col + j);
                                    ++sc;
                                    if (ldcg_i(dr + p) != l - 1) continue;
                                    const double sp = ldcg_d2(sdr + p).x;
                                    atomicAdd(dacc + p, __dmul_rn(__ddiv_rn(sp, sx), g));
                                    by += 24;
                                    if (atomicMax(mark + p, mU) < E) Unext[append_smem(&s_ucnt)] = p;
                                }
                            }
                            group_sync<G>();
                            if (gl == 0) {
                                dacc[x] = 0.0;
                                sdr[x].y = ldcg_d2(sdr + x).y + g;
                                atomicAdd(a.bc + x, g);
                                by += 8 + 8 + 16 + 16 + (r.y > r.x ? 8 : 0);
                            }
                            st_bytes += by + 8 * sc;
                            st_scanned += sc;
                        });
                    // removal-push targets at level l
                    if (rcnt) {
                        two_tier(
                            rcnt, a.g, lim,
                            [&](int i, int &x) { x = Rv[i]; return Rl[i] == l; },
                            [&](int, int) { return l >= 2; },
                            [&](auto Gc, int, int x, int2 r, int gl) {
                                constexpr int G = decltype(Gc)::value;
                                const double g = ldcg_d(dacc + x);
                                unsigned long long by = 0, sc = 0;
                                if (g != 0.0) {
                                    const double sx = ldcg_d2(sdr + x).x;
                                    for (int j = r.x + gl; j < r.y; j += G) {
                                        const int p = ldg_i(a.g.col + j);
                                        ++sc;
                                        if (ldcg_i(dr + p) != l - 1) continue;
                                        const double sp = ldcg_d2(sdr + p).x;
                                        atomicAdd(dacc + p, __dmul_rn(__ddiv_rn(sp, sx), g));
                                        by += 24;
                                        if (atomicMax(mark + p, mU) < E) Unext[append_smem(&s_ucnt)] = p;
                                    }
                                }
                                group_sync<G>();
                                if (gl == 0) {
                                    dacc[x] = 0.0;
                                    sdr[x].y = ldcg_d2(sdr + x).y + g;
                                    atomicAdd(a.bc + x, g);
                                    by += 8 + 8 + 16 + 16 + (r.y > r.x ? 8 : 0);
                                }
                                st_bytes += by + 8 * sc;
                                st_scanned += sc;
                            });
                    }
                    __syncthreads();
                    ucnt = s_ucnt;
                    __syncthreads();
                    if (tid == 0) {
                        s_ucnt = 0;
                        st_touched += ucnt;
                    }
                    int *t = Ucur;
                    Ucur = Unext;
                    Unext = t;
                    __syncthreads();
                }
                // any up vertices left at level 0 would be the root: never produced
                if (case3) {  // distances changed: re-classify from the next insertion
                    ++p;
                    break;
                }
            }
            ins = p;
            __syncthreads();  // s_work is rewritten by the next window
        }
    }
    if (tid == 0) {
        a.ws.wepoch[wk] = epoch;
        if (st_case[0]) atomicAdd(a.stats + kStCase1, st_case[0]);
        if (st_case[1]) atomicAdd(a.stats + kStCase2, st_case[1]);
        if (st_case[2]) atomicAdd(a.stats + kStCase3, st_case[2]);
        if (st_touched) atomicAdd(a.stats + kStTouched, st_touched);
        if (st_down) atomicAdd(a.stats + kStDown, st_down);
    }
    if (st_scanned) atomicAdd(a.stats + kStScanned, st_scanned);
    if (st_bytes) atomicAdd(a.stats + kStBytes, st_bytes);
}

void launch_update(const UpdateArgs &a, int workers, cudaStream_t s) {
    update_kernel<<<workers, kBlock, 0, s>>>(a);
}

}  // namespace dbc
