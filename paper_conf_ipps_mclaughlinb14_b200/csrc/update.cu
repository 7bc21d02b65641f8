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

// per-phase timers (diagnostic; %globaltimer reads sit on thread 0's critical
// path, so they are compiled in only with -DDBC_PHASE_TIMERS)
#ifdef DBC_PHASE_TIMERS
constexpr bool kPhaseTimers = true;
#else
constexpr bool kPhaseTimers = false;
#endif

namespace {
// Dold[i] = old level of D[i] (low 31 bits) | kExtPred if D[i] has a predecessor
// outside D (only such rows push in the up phase)
constexpr int32_t kOldMask = 0x7fffffff;
constexpr int32_t kExtPred = INT32_MIN;

// A C2 push pass: flat_entries (dbc_internal.cuh) whose visitor f(t, y, d, sd,
// mark) returns the mark to claim y with (0: none); the claims of a thread's
// kFlatU entries are issued together -- one atomic round trip instead of one
// per entry -- and onclaim(y) runs for each vertex this thread claimed.
template <bool kCG, class Want, class Col, class F, class OnClaim>
__device__ __forceinline__ void flat_push(const int *off, int cnt, int E, Col colf, const Root &st,
                                          uint32_t *mk, uint32_t Etag, Want want, F f, OnClaim onclaim,
                                          int Ebeg = 0) {
    const int tid = threadIdx.x;
    for (int base = Ebeg; base < E; base += kBlock * kFlatU) {
        const int e0 = base + tid * kFlatU;
        int t[kFlatU], y[kFlatU], dy[kFlatU];
        uint32_t mm[kFlatU], req[kFlatU];
        int cur = -1;
        if (e0 < E) {
            int lo = 0, hi = cnt - 1;  // last row with off[row] <= e0
            while (lo < hi) {
                const int mid = (lo + hi + 1) >> 1;
                if (off[mid] <= e0) lo = mid; else hi = mid - 1;
            }
            cur = lo;
        }
#pragma unroll
        for (int u = 0; u < kFlatU; ++u) {
            const int e = e0 + u;
            t[u] = -1;
            y[u] = 0;
            if (e < E) {
                while (off[cur + 1] <= e) ++cur;
                t[u] = cur;
                y[u] = colf(cur, e);
            }
        }
#pragma unroll
        for (int u = 0; u < kFlatU; ++u)
            dy[u] = (t[u] >= 0) ? (kCG ? __ldcg(st.d + y[u]) : st.dist(y[u])) : kInf;
#pragma unroll
        for (int u = 0; u < kFlatU; ++u)
            mm[u] = (t[u] >= 0 && want(dy[u])) ? (kCG ? __ldcg(mk + y[u]) : mk[y[u]]) : 0u;
#pragma unroll
        for (int u = 0; u < kFlatU; ++u) req[u] = (t[u] >= 0) ? f(t[u], y[u], dy[u], mm[u]) : 0u;
        uint32_t prev[kFlatU];
#pragma unroll
        for (int u = 0; u < kFlatU; ++u) prev[u] = req[u] ? atomicMax(mk + y[u], req[u]) : 0xffffffffu;
#pragma unroll
        for (int u = 0; u < kFlatU; ++u)
            if (prev[u] < Etag) onclaim(y[u]);
    }
    __syncthreads();
}

// One push of a helped C2 pass (owner or helper): the same arithmetic as the
// owner's up_visit / dpush_visit; returns the claim request (flat_push issues
// it and appends the claimed vertex to the global list).
__device__ __forceinline__ uint32_t help_push_entry(const GView &g, const ChunkSmem &M, int t, int pp, int dp,
                                                    uint32_t mp, const HelpCtx &cx, double *dacc,
                                                    uint32_t &bytes) {
    if (dp != cx.l - 1) return 0u;
    const uint32_t E = cx.E, mD = E | kDown, mU = E | kUp;
    const int meta = M.meta[t];
    double dlt;  // Ddelta[p] / sigma[p] (the accumulator is sigma-factored)
    if (meta & kMetaUp) {
        dlt = __ddiv_rn(M.c1[t], M.c0[t]);
    } else {
        if (mp == mD) return 0u;
        dlt = __ddiv_rn(1.0 + M.acc[t], M.c0[t]);
        if ((meta & kMetaNotPulled) && !((meta & kMetaNew) && new_edge(g, M.v[t], pp, cx.g0, cx.lim)))
            dlt = __dsub_rn(dlt, __ddiv_rn(1.0 + M.c1[t], M.c2[t]));
    }
    atomicAdd(dacc + pp, dlt);
    bytes += 24;
    return mp >= E ? 0u : mU;
}

// Entries [e0, e1) of a published chunk M (in this CTA's shared memory).
// kCG: the owner's state is read through L2 (helpers run on other SMs).
template <bool kCG>
__device__ __forceinline__ void help_run_block(const ChunkSmem &M, int e0, int e1, const GView &g,
                                               const Root &st, uint32_t *mark, double *dacc, int32_t *gU,
                                               int *gapp, const HelpCtx &cx, uint32_t &bytes) {
    auto colf = [&](int t, int e) { return ldg_i(g.col + M.beg[t] + e - M.off[t]); };
    flat_push<kCG>(
        M.off, cx.cnt, e1, colf, st, mark, cx.E, [&](int dp) { return dp == cx.l - 1; },
        [&](int t, int pp, int dp, uint32_t mp) -> uint32_t {
            if (M.meta[t] & kMetaUp) bytes += 8;  // D rows: counted by their C1 pull
            return help_push_entry(g, M, t, pp, dp, mp, cx, dacc, bytes);
        },
        [&](int pp) { gU[atomicAdd(gapp, 1)] = pp; }, e0);
}

// ---------------------------------------------------------------------------
// One level of the down phase (K3) over items [i0, i1) of the level -- the
// owner's whole level, or one block of a helped level (owner or helper CTA).
struct DownCtx {
    GView g;
    Root st;
    uint32_t *mark;
    unsigned long long *lowrec;
    int32_t *Dv, *Dold;
    double *Dsig;
    uint32_t *mask;   // the root's level-2 predecessor masks
    int32_t *err;
    int *dcnt;        // D append counter (shared; global on a helped level)
    int *lowflag;     // set when a distance is lowered (Case 3)
    const int *adjs;  // the root's row (bit positions of the masks), dsr entries
    int dsr, L, lb, lim, mvalid, del;
    uint32_t epoch, mD;
};
// helped down levels: UpdateArgs.hd_min items at least, hd_block items per block

__device__ __forceinline__ uint32_t dc_l1bit(const DownCtx &c, int y) {
    for (int j = 0; j < c.dsr; ++j)
        if (c.adjs[j] == y) return 1u << j;
    return 0u;
}

// per-D-entry epilogue: record old d / sigma, store the new sigma (and, at
// level 2, the vertex's level-1 predecessor mask)
__device__ __forceinline__ void dc_finish(const DownCtx &c, int idx, int w, double sum, uint32_t m, bool ext,
                                          uint32_t &bytes) {
    if (c.mvalid && c.L == 2) c.mask[w] = m;
    const unsigned long long lr = c.lowrec[w];
    const int od = ((uint32_t)(lr >> 32) == c.epoch) ? (int)(uint32_t)lr : c.L;
    c.Dold[idx] = od | (ext ? kExtPred : 0);
    c.Dsig[idx] = c.st.sd[w].x;
    c.st.sd[w].x = sum;
    if (!(sum <= 1.7976931348623157e308)) atomicOr(c.err, kErrNumeric);
    bytes += 8 + 8 + 20;
}

// one neighbour y of a level-L vertex; returns sigma[y] if y is a predecessor
__device__ __forceinline__ double dc_visit(const DownCtx &c, int y, int dy, double sy, uint32_t &bytes) {
    const int L = c.L;
    if (dy == L - 1) {
        bytes += 8;
        return sy;
    }
    if (dy > L + 1) {  // Case 3 pull-up
        const int old = atomicMin(c.st.d + y, L + 1);
        if (old > L + 1 && !(c.del && (uint32_t)(c.lowrec[y] >> 32) == c.epoch)) {
            c.lowrec[y] = ((unsigned long long)c.epoch << 32) | (uint32_t)old;
            *c.lowflag = 1;
            bytes += 4;
        }
        dy = L + 1;
    }
    if (dy == L + 1 && atomicMax(c.mark + y, c.mD) < c.mD) c.Dv[atomicAdd(c.dcnt, 1)] = y;
    return 0.0;
}

// short rows of items [i0, i1) walked in-lane in canonical order (bit-exact
// sigma); long rows handed to enq(item, length)
template <class Enq>
__device__ __forceinline__ void dc_small(const DownCtx &c, int i0, int i1, Enq enq, uint32_t &bytes,
                                         uint32_t &scanned) {
    const int L = c.L, mD = c.mD;
    for (int i = i0 + (int)threadIdx.x; i < i1; i += kBlock) {
        const int w = c.Dv[c.lb + i];
        const int2 r = row_of(c.g, w, c.lim);
        if (r.y - r.x > kSmallDeg) {
            enq(i, r.y - r.x);
            continue;
        }
        double sum = 0.0;  // canonical order: bit-exact
        uint32_t m = 0u;
        bool ext = false;
        for (int j = r.x; j < r.y; j += kRowUnroll) {
            int y[kRowUnroll], dy[kRowUnroll], om[kRowUnroll];
            uint32_t oc[kRowUnroll], pm[kRowUnroll];
            double sy[kRowUnroll];
#pragma unroll
            for (int u = 0; u < kRowUnroll; ++u) y[u] = (j + u < r.y) ? ldg_i(c.g.col + j + u) : -1;
#pragma unroll
            for (int u = 0; u < kRowUnroll; ++u) dy[u] = (y[u] >= 0) ? c.st.d[y[u]] : kInf;
#pragma unroll
            for (int u = 0; u < kRowUnroll; ++u) {
                const bool pr = y[u] >= 0 && dy[u] == L - 1;
                sy[u] = pr ? c.st.sd[y[u]].x : 0.0;
                pm[u] = pr ? c.mark[y[u]] : (uint32_t)mD;
            }
            // issue every lowering and claim of the block, then consume
#pragma unroll
            for (int u = 0; u < kRowUnroll; ++u)
                om[u] = (y[u] >= 0 && dy[u] > L + 1) ? atomicMin(c.st.d + y[u], L + 1) : 0;
#pragma unroll
            for (int u = 0; u < kRowUnroll; ++u) oc[u] = mD;
#pragma unroll
            for (int u = 0; u < kRowUnroll; ++u)
                if (y[u] >= 0 && dy[u] >= L + 1) oc[u] = atomicMax(c.mark + y[u], (uint32_t)mD);
#pragma unroll
            for (int u = 0; u < kRowUnroll; ++u) {
                if (y[u] < 0) continue;
                if (dy[u] == L - 1) {  // predecessor: canonical-order sum
                    sum += sy[u];
                    ext |= pm[u] != (uint32_t)mD;
                    bytes += 8;
                    if (c.mvalid && L == 2) m |= dc_l1bit(c, y[u]);
                }
                if (dy[u] > L + 1 && om[u] > L + 1 &&  // first lowerer (Case 3)
                    !(c.del && (uint32_t)(c.lowrec[y[u]] >> 32) == c.epoch)) {
                    c.lowrec[y[u]] = ((unsigned long long)c.epoch << 32) | (uint32_t)om[u];
                    *c.lowflag = 1;
                    bytes += 4;
                }
                if (dy[u] >= L + 1 && oc[u] < (uint32_t)mD) c.Dv[atomicAdd(c.dcnt, 1)] = y[u];
            }
        }
        bytes += 8 + 8ull * (r.y - r.x);
        scanned += r.y - r.x;
        dc_finish(c, c.lb + i, w, sum, m, ext, bytes);
    }
}

// the long rows queued in Bq[0, nbig) (item indices), kBig per round through
// S, entries flattened over the CTA.  Caller: barrier before (queue complete);
// ends with a barrier.
__device__ __forceinline__ void dc_big(const DownCtx &c, BigSmem &S, const int32_t *Bq, int nbig,
                                       uint32_t &bytes, uint32_t &scanned) {
    const int tid = threadIdx.x, L = c.L;
    for (int r0 = 0; r0 < nbig; r0 += kBig) {
        const int m = min(kBig, nbig - r0);
        big_load(S, m, [&](int t) { return Bq[r0 + t]; }, [&](int i) { return c.Dv[c.lb + i]; }, c.g, c.lim);
        if (tid < m) {
            S.mk[tid] = 0u;
            S.ext[tid] = 0;
        }
        __syncthreads();
        big_entries(S, c.g, c.st, [&](int dy) { return dy == L - 1; }, [&](int t, int y, int dy, double2 q) {
            bytes += 8;
            scanned++;
            if (c.mvalid && L == 2 && dy == 1) atomicOr(&S.mk[t], dc_l1bit(c, y));
            if (dy == L - 1 && c.mark[y] != c.mD) S.ext[t] = 1;
            return dc_visit(c, y, dy, q.x, bytes);
        });
        if (tid < m) {
            double sum = S.acc[tid];
            const int w = S.v[tid];
            if (sum >= kExact) {  // order-dependent rounding: canonical sum
                const int2 r = row_of(c.g, w, c.lim);
                sum = 0.0;
                for (int j = r.x; j < r.y; ++j) {
                    const int y = ldg_i(c.g.col + j);
                    if (c.st.dist(y) == L - 1) sum += c.st.sd[y].x;
                }
            }
            bytes += 8;
            dc_finish(c, c.lb + S.idx[tid], w, sum, S.mk[tid], S.ext[tid] != 0, bytes);
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------
// (0) Case-3 removal pushes (A4 step 0) over D items [i0, i1): every pulled-up
// w (finite old level od != d[w]) gives each old predecessor x outside D
//   Ddelta[x] -= sigma[x] / sigma_old(w) * (1 + delta_old(w))
// (the accumulator holds Ddelta / sigma: DESIGN.md Sec. 6), and x becomes an
// up vertex of level od - 1.  The owner's whole pass, or one block of a helped
// pass (then rcnt / rmax are the owner's global counters).  Ends with a barrier.
struct RemCtx {
    GView g;
    Root st;
    uint32_t *mark;
    double *dacc;
    const int32_t *Dv, *Dold;
    const double *Dsig;
    int32_t *Rv, *Rl;
    int *rcnt, *rmax;
    int g0, lim;
    uint32_t E, mD, mU;
};

__device__ __forceinline__ void rem_visit(const RemCtx &c, int w, int od, double osig, double coef, int x,
                                          int dx, uint32_t &bytes) {
    if (dx != od - 1) return;
    if (c.mark[x] == c.mD) return;
    if (ldg_i(c.g.rp + w) < 0 && new_edge(c.g, w, x, c.g0, c.lim)) return;  // not an old predecessor
    atomicAdd(c.dacc + x, -__ddiv_rn(coef, osig));
    bytes += 24;
    if (atomicMax(c.mark + x, c.mU) < c.E) {
        const int pos = atomicAdd(c.rcnt, 1);
        c.Rv[pos] = x;
        c.Rl[pos] = od - 1;
        atomicMax(c.rmax, od - 1);
    }
}

__device__ __forceinline__ void rem_range(const RemCtx &c, BigSmem &S, int *s_old, int32_t *Bq, int *nbig,
                                          int i0, int i1, uint32_t &bytes,
                                          uint32_t &scanned) {
    const int tid = threadIdx.x;
    split_pass(
        i1 - i0, c.g, c.lim,
        [&](int q, int &w) {
            const int i = i0 + q;
            const int od = c.Dold[i] & kOldMask;
            w = c.Dv[i];
            return od != kInf && od != c.st.dist(w);
        },
        [&](int q, int w, int2 r) {
            const int i = i0 + q;
            const int od = c.Dold[i] & kOldMask;
            const double osig = c.Dsig[i];
            const double coef = 1.0 + c.st.sd[w].y;  // delta still old
            row_walk(c.g, c.st, nullptr, r, [&](int dx) { return dx == od - 1; },
                     [&](int x, int dx, double2, uint32_t) { rem_visit(c, w, od, osig, coef, x, dx, bytes); });
            bytes += 8 + 8ull * (r.y - r.x);
            scanned += r.y - r.x;
        },
        [&](int q) { Bq[atomicAdd(nbig, 1)] = i0 + q; });
    __syncthreads();
    const int nb = *nbig;
    for (int r0 = 0; r0 < nb; r0 += kBig) {
        const int m = min(kBig, nb - r0);
        big_load(S, m, [&](int t) { return Bq[r0 + t]; }, [&](int i) { return c.Dv[i]; }, c.g, c.lim);
        if (tid < m) {
            const int i = S.idx[tid];
            S.c0[tid] = c.Dsig[i];
            s_old[tid] = c.Dold[i] & kOldMask;  // old level of each row
            bytes += 8;
        }
        __syncthreads();
        big_entries(S, c.g, c.st, [](int) { return true; }, [&](int t, int x, int dx, double2) {
            bytes += 8;
            scanned++;
            const int w = S.v[t];
            rem_visit(c, w, s_old[t], S.c0[t], 1.0 + c.st.sd[w].y, x, dx, bytes);
            return 0.0;
        });
    }
    __syncthreads();
    if (tid == 0) *nbig = 0;
    __syncthreads();
}

// ---------------------------------------------------------------------------
// Long rows of a down level, entry-balanced (a level's long rows can hold most
// of its entries -- hub neighbourhoods -- so blocks of rows would not balance).
// The owner queues the level's long rows (item indices) in Bq[0, nrows), builds
// exclusive entry offsets Boff[0..nrows] (dl_offsets), then the entries are
// processed in blocks of he_entries (dl_block, owner and helpers): per entry the
// down-phase visit (lowering, claims), per row the predecessor-sigma partial sum
// added into dacc[w] (sums of integer-valued sigma: exact in any order below
// 2^53, else the owner re-sums the row in canonical order), the "predecessor
// outside D" flag as bit 31 of Bq[t], and level-2 mask bits into mask[w].
// dl_finish (owner) completes every row with dc_finish.
constexpr uint32_t kBqExt = 0x80000000u;
constexpr int kDlEntries = 32 * kBig;  // entries per block: spans <= kBig long rows (> kSmallDeg entries each)

// owner: offsets of Bq[0, nrows) into Boff (uses I.off as scratch); returns the
// entry total (every thread).  Ends with a barrier.
__device__ __forceinline__ int dl_offsets(const DownCtx &c, int32_t *Bq, int32_t *Boff, int nrows, int *soff,
                                          int *s_tot) {
    const int tid = threadIdx.x;
    if (tid == 0) *s_tot = 0;
    __syncthreads();
    for (int r0 = 0; r0 < nrows; r0 += kChunk) {
        const int m = min(kChunk, nrows - r0);
        for (int i = tid; i < m; i += kBlock) {
            const int w = c.Dv[c.lb + Bq[r0 + i]];
            const int2 r = row_of(c.g, w, c.lim);
            soff[i + 1] = r.y - r.x;
            if (c.mvalid && c.L == 2) c.mask[w] = 0u;
        }
        __syncthreads();
        chunk_scan(soff, m);  // ends with a barrier
        const int carry = *s_tot;
        for (int i = tid; i < m; i += kBlock) Boff[r0 + i] = carry + soff[i];
        __syncthreads();
        if (tid == 0) *s_tot = carry + soff[m];
        __syncthreads();
    }
    const int tot = *s_tot;
    if (tid == 0) Boff[nrows] = tot;
    return tot;
}

// entries [e0, e1) of the published long rows (owner or helper; kCG: read the
// owner's lists through L2).  Ends with a barrier.
template <bool kCG>
__device__ __forceinline__ void dl_block(const DownCtx &c, BigSmem &S, int32_t *Bq, const int32_t *Boff,
                                         int nrows, int e0, int e1, double *dacc, int *s_t0,
                                         uint32_t &bytes, uint32_t &scanned) {
    const int tid = threadIdx.x, L = c.L;
    // first row: last t with Boff[t] <= e0 (two strided probes over the CTA)
    if (tid == 0) *s_t0 = 0;
    __syncthreads();
    const int stride = (nrows + kBlock - 1) / kBlock;
    {
        const int t = tid * stride;
        if (t < nrows && (kCG ? __ldcg(Boff + t) : Boff[t]) <= e0) atomicMax(s_t0, tid);
    }
    __syncthreads();
    const int j0 = *s_t0 * stride;
    __syncthreads();
    if (tid < stride && j0 + tid < nrows && (kCG ? __ldcg(Boff + j0 + tid) : Boff[j0 + tid]) <= e0)
        atomicMax(s_t0, j0 + tid);
    __syncthreads();
    const int t0 = *s_t0;
    // rows t0 .. (at most kBig of them: long rows have > kSmallDeg entries)
    if (tid < kBig) {
        const int t = t0 + tid;
        const int bo = (t < nrows) ? (kCG ? __ldcg(Boff + t) : Boff[t]) : e1;
        if (bo < e1) {
            const int idx = (int)((uint32_t)(kCG ? __ldcg(Bq + t) : Bq[t]) & ~kBqExt);
            const int w = kCG ? __ldcg(c.Dv + c.lb + idx) : c.Dv[c.lb + idx];
            const int2 r = row_of(c.g, w, c.lim);
            S.v[tid] = w;
            S.b[tid] = r.x;
            S.off[tid] = bo;
            S.acc[tid] = 0.0;
            S.mk[tid] = 0u;
            S.ext[tid] = 0;
            S.idx[tid] = 1;
        } else {
            S.idx[tid] = 0;
        }
    }
    __syncthreads();
    if (tid < kBig && S.idx[tid] && (tid + 1 == kBig || !S.idx[tid + 1])) S.m = tid + 1;
    __syncthreads();
    const int m = S.m;
    for (int base = e0; base < e1; base += kUnroll * kBlock) {
        int t[kUnroll], y[kUnroll], dy[kUnroll];
        double sy[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
            const int e = base + u * kBlock + tid;
            t[u] = -1;
            y[u] = 0;
            if (e < e1) {
                int lo = 0, hi = m - 1;  // last row with off <= e
                while (lo < hi) {
                    const int mid = (lo + hi + 1) >> 1;
                    if (S.off[mid] <= e) lo = mid; else hi = mid - 1;
                }
                t[u] = lo;
                y[u] = ldg_i(c.g.col + S.b[lo] + (e - S.off[lo]));
            }
        }
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) dy[u] = (t[u] >= 0) ? (kCG ? __ldcg(c.st.d + y[u]) : c.st.dist(y[u])) : kInf;
#pragma unroll
        for (int u = 0; u < kUnroll; ++u)
            sy[u] = (t[u] >= 0 && dy[u] == L - 1) ? (kCG ? __ldcg(&c.st.sd[y[u]].x) : c.st.sd[y[u]].x) : 0.0;
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
            double cc = 0.0;
            if (t[u] >= 0) {
                bytes += 8;
                scanned++;
                if (dy[u] == L - 1) {
                    if (c.mvalid && L == 2) atomicOr(&S.mk[t[u]], dc_l1bit(c, y[u]));
                    if ((kCG ? __ldcg(c.mark + y[u]) : c.mark[y[u]]) != c.mD) S.ext[t[u]] = 1;
                }
                cc = dc_visit(c, y[u], dy[u], sy[u], bytes);
            }
            acc_add(S.acc, t[u], cc);
        }
    }
    __syncthreads();
    if (tid < m) {  // publish the block's per-row partials
        const int w = S.v[tid];
        if (S.acc[tid] != 0.0) atomicAdd(dacc + w, S.acc[tid]);
        if (S.ext[tid]) atomicOr((uint32_t *)(Bq + t0 + tid), kBqExt);
        if (S.mk[tid]) atomicOr(c.mask + w, S.mk[tid]);
    }
    __syncthreads();
}

// owner: complete the long rows after every block ran
__device__ __forceinline__ void dl_finish(const DownCtx &c, const int32_t *Bq, int nrows, double *dacc,
                                          uint32_t &bytes) {
    const int L = c.L;
    for (int t = threadIdx.x; t < nrows; t += kBlock) {
        const uint32_t q = (uint32_t)__ldcg(Bq + t);
        const int idx = (int)(q & ~kBqExt);
        const int w = c.Dv[c.lb + idx];
        double sum = __ldcg(dacc + w);
        dacc[w] = 0.0;
        if (sum >= kExact) {  // order-dependent rounding: canonical sum
            const int2 r = row_of(c.g, w, c.lim);
            sum = 0.0;
            for (int j = r.x; j < r.y; ++j) {
                const int y = ldg_i(c.g.col + j);
                if (c.st.dist(y) == L - 1) sum += c.st.sd[y].x;
            }
        }
        const uint32_t m = (c.mvalid && L == 2) ? __ldcg(c.mask + w) : 0u;
        dc_finish(c, c.lb + idx, w, sum, m, (q & kBqExt) != 0, bytes);
    }
    __syncthreads();
}

// ---------------------------------------------------------------------------
// The in-lane item pass of a wide up level as help blocks (kind 5): items
// [q0, q1) of level l -- the down segment Dv[b0, b0 + nDl), then the up
// frontier (Ul / Uo), then removal targets of level l -- resolved and, for
// short rows, processed in-lane exactly as the owner's inlane() does (delta
// pull of down rows, Ddelta pushes to level l - 1, Alg. 8 epilogue); long rows
// are deferred to the owner's X list (its chunks run after the pass).  Claimed
// predecessors are appended to gU.  Owner and helpers run the same code.
struct UpCtx {
    GView g;
    Root st;
    uint32_t *mark;
    double *dacc, *bc;
    const uint32_t *mask;
    const int32_t *Dv, *Dold, *Rv, *Rl, *Ul, *Uo;
    const double *Dsig;
    const int *adjs;  // the root's row (level-2 mask bits)
    int32_t *gU;
    int *gapp, *xcnt;
    XRow *X;
    int l, b0, nDl, ucnt, g0, lim, mok;
    uint32_t E, mU, mD;
};

__device__ __forceinline__ void up_claim(const UpCtx &c, int y, uint32_t my) {
    if (my >= c.E) return;
    if (atomicMax(c.mark + y, c.mU) >= c.E) return;
    c.gU[atomicAdd(c.gapp, 1)] = y;
}

__device__ __forceinline__ void up_block(const UpCtx &c, int q0, int q1, uint32_t &bytes, uint32_t &scanned) {
    const int l = c.l;
    const bool push = l >= 2;
    for (int q = q0 + (int)threadIdx.x; q < q1; q += kBlock) {
        // ---- resolve (as the owner's resolve())
        int x, meta;
        double c0, c1, c2;
        int2 r;
        uint32_t mk = 0u;
        if (q < c.nDl) {
            const int idx = c.b0 + q;
            x = c.Dv[idx];
            const double2 s2 = c.st.sd[x];
            c0 = s2.x;
            c1 = s2.y;
            c2 = c.Dsig[idx];
            const int od = c.Dold[idx];
            meta = (((od & kOldMask) == l) ? kMetaNotPulled : 0) | ((od < 0) ? kMetaExt : 0) |
                   ((ldg_i(c.g.rp + x) < 0) ? kMetaNew : 0);
            r = row_of(c.g, x, c.lim);
            bytes += 8 + 8;
        } else {
            const int qi = q - c.nDl;
            x = -1;
            if (qi < c.ucnt)
                x = (qi < kUcap) ? c.Ul[qi] : c.Uo[qi - kUcap];
            else if (c.Rl[qi - c.ucnt] == l)
                x = c.Rv[qi - c.ucnt];
            if (x < 0) continue;
            const uint32_t prev = atomicMax(c.mark + x, c.E | kUpDone);
            const double gxs = __ldcg(c.dacc + x);
            const double2 s2 = c.st.sd[x];
            const double sx = s2.x, odl = s2.y;
            const double gx = __dmul_rn(sx, gxs);
            const bool usemask = l == 2 && c.mok;
            const int2 rr = (push && !usemask) ? row_of(c.g, x, c.lim) : make_int2(0, 0);
            mk = usemask ? c.mask[x] : 0u;
            if (prev != c.mU) continue;  // a duplicate: the first claimant processes
            meta = kMetaUp | (usemask ? kMetaMask : 0);
            c0 = sx;
            c1 = gx;
            c2 = odl;
            bytes += 8 + (usemask ? 4 : 0);
            r = (push && gx != 0.0) ? rr : make_int2(0, 0);
            if (gx == 0.0) mk = 0u;
        }
        const int len = r.y - r.x;
        if (len > kSmallDeg) {  // long row: a deferred chunk of the owner
            const bool up = (meta & kMetaUp) != 0;
            const int xi = atomicAdd(c.xcnt + (up ? 1 : 0), 1);
            if (xi < kXcap / 2) {
                XRow &w = c.X[up ? kXcap - 1 - xi : xi];
                w.x = x;
                w.meta = meta;
                w.beg = r.x;
                w.len = len;
                w.c0 = c0;
                w.c1 = c1;
                w.c2 = c2;
                w.mk = mk;
                continue;
            }
            // list full: walk it here
        }
        // ---- in-lane (as the owner's inlane())
        const bool wantpush = push && r.y > r.x;
        if (meta & kMetaMask) {  // level 2: predecessors = set bits (root's row order)
            for (uint32_t b = mk; b; b &= b - 1) {
                const int pp = c.adjs[__ffs(b) - 1];
                atomicAdd(c.dacc + pp, __ddiv_rn(c1, c0));
                bytes += 24;
                up_claim(c, pp, c.mark[pp]);
            }
        } else if (meta & kMetaUp) {
            if (wantpush) {
                const double wx = __ddiv_rn(c1, c0);  // Ddelta[x] / sigma[x]
                for (int j = r.x; j < r.y; j += kRowUnroll) {
                    int y[kRowUnroll], dy[kRowUnroll];
                    uint32_t mp[kRowUnroll];
#pragma unroll
                    for (int u = 0; u < kRowUnroll; ++u) y[u] = (j + u < r.y) ? ldg_i(c.g.col + j + u) : -1;
#pragma unroll
                    for (int u = 0; u < kRowUnroll; ++u) dy[u] = (y[u] >= 0) ? c.st.d[y[u]] : kInf;
#pragma unroll
                    for (int u = 0; u < kRowUnroll; ++u) mp[u] = (y[u] >= 0 && dy[u] == l - 1) ? c.mark[y[u]] : 0xffffffffu;
#pragma unroll
                    for (int u = 0; u < kRowUnroll; ++u)
                        if (y[u] >= 0 && dy[u] == l - 1) {
                            atomicAdd(c.dacc + y[u], wx);
                            bytes += 24;
                            up_claim(c, y[u], mp[u]);
                        }
                }
                scanned += r.y - r.x;
                bytes += 8 + 8u * (r.y - r.x);
            }
        } else {
            double dn = 0.0;
            row_walk(c.g, c.st, nullptr, r, [&](int dy) { return dy == l + 1; },
                     [&](int, int dy, double2 qq, uint32_t) {
                         if (dy == l + 1) {
                             bytes += 16;
                             dn += __dmul_rn(__ddiv_rn(c0, qq.x), __dadd_rn(1.0, qq.y));
                         }
                     });
            scanned += r.y - r.x;
            bytes += 8u * (r.y - r.x);
            if (wantpush && (meta & kMetaExt)) {  // some predecessor outside D
                row_walk(c.g, c.st, c.mark, r, [&](int dp) { return dp == l - 1; },
                         [&](int pp, int dp, double2, uint32_t mp) {
                             if (dp != l - 1 || mp == c.mD) return;
                             double dlt = __ddiv_rn(1.0 + dn, c0);
                             if ((meta & kMetaNotPulled) &&
                                 !((meta & kMetaNew) && new_edge(c.g, x, pp, c.g0, c.lim)))
                                 dlt = __dsub_rn(dlt, __ddiv_rn(1.0 + c1, c2));
                             atomicAdd(c.dacc + pp, dlt);
                             bytes += 24;
                             up_claim(c, pp, mp);
                         });
                scanned += r.y - r.x;
                (void)0;  // the second walk of the row: one pass in the byte model
            }
            c.st.sd[x].y = dn;  // d_finish
            atomicAdd(c.bc + x, dn - c1);
            bytes += 8 + 16;  // delta write, BC RMW
            continue;
        }
        // up_finish
        c.dacc[x] = 0.0;
        c.st.sd[x].y = c2 + c1;
        atomicAdd(c.bc + x, c1);
        bytes += 16 + 16;  // delta RMW, BC RMW
    }
    __syncthreads();
}

__global__ void __launch_bounds__(kBlock, kMinBlocks) update_kernel(UpdateArgs a) {
    __shared__ int s_slot;
    __shared__ int s_dcnt;     // |D| (absolute positions in Dv)
    __shared__ int s_ucnt2[2]; // up frontier sizes (list ucur_sel is read, ucur_sel^1 filled)
    __shared__ int s_rcnt;     // |R|
    __shared__ int s_rmax;     // deepest removal-push target level
    __shared__ int s_nbig;     // long-row queue (down phase / removal)
    __shared__ int s_nbigI;    // long rows of the current up level (in I)
    __shared__ int s_noext;    // the chunk holds down rows without pushes
    __shared__ int s_nl1;      // of those, resolved against adj(root)
    __shared__ int s_ds;       // |adj(root)| as of the insertion (-1: too long)
    __shared__ int s_wcnt[2];            // window: insertions with work, of which Case 3
    __shared__ int s_job[8];             // [2] lowest seed level, [3] any lowering, [4] mask state, [5] root degree, [7] deepest seed level
    __shared__ BigSmem S;
    __shared__ ChunkSmem I;              // long rows of the current up level
    __shared__ int s_l1[kChunk];
    __shared__ int s_adjs[kAdjCap];      // adj(root) = the level-1 vertices
    __shared__ int s_adjdeg[kAdjCap];    // their degrees
    __shared__ double s_l1acc[kAdjCap];  // per level-1 vertex: sum of Ddelta[x] / sigma[x]
    __shared__ int s_un[2][kUcap];       // up frontier ping-pong (overflow: U0 / U1)
    __shared__ int s_hb, s_hpick, s_hseq; // cooperative help: grabbed block, owner, request
    __shared__ HelpCtx s_hctx;
    __shared__ int s_hadjs[kMaskDeg], s_hds;  // helped down level: the owner's root row (mask bits)
    __shared__ int s_hopen;                   // open requests seen at the last level boundary
    __shared__ int s_nent, s_tot, s_t0;        // long rows of a down level: entries, offsets total, first row
    __shared__ int s_stg[3];                  // helped down block: staged long rows, their entries, base
    __shared__ int s_nx[2];                   // wide up level: deferred long down / up rows
    __shared__ int s_del[6];     // deletion job: [0] u_high, [1] u_low, [2] |A|, [3] seeds, [4] candidates, [5] u_low keeps a predecessor
    __shared__ double s_delsd[2];  // deletion job: old sigma / delta of u_low

    const int tid = threadIdx.x;
    const int wk = a.worker_base + blockIdx.x;  // scratch of this worker
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
    int32_t *Bq = a.ws.Bq + (size_t)wk * n;
    int32_t *Wul = a.ws.Wul + (size_t)wk * a.ws.wcap;    // window: u_low of each insertion
    int32_t *Wlev = a.ws.Wlev + (size_t)wk * a.ws.wcap;  // window: seed level d[u_high] + 1 (INT32_MAX: Case 1)
    uint32_t epoch = a.ws.wepoch[wk];
    const GView &g = a.g;
    int hseq = 0;  // this worker's help-request sequence

    // diagnostic counters: per-thread bytes / entries scanned in 32 bits (one
    // launch moves < 4 GB per thread), thread 0's tallies in shared memory --
    // registers are the occupancy limit of this kernel
    uint32_t st_bytes = 0;
    uint32_t sc_down = 0, sc_rem = 0, sc_dpull = 0, sc_dpush = 0, sc_up2 = 0, sc_up3 = 0;
    __shared__ unsigned long long s_st[7];    // touched, down, case 1/2/3, level steps down/up (thread 0)
    __shared__ unsigned long long s_touch0;   // touched count at the job start (scenario log)
    __shared__ unsigned long long s_prof[5];  // root profile: t0, jobs, touched0, scanned0, levels0 (thread 0)
    if (tid == 0)
        for (int q = 0; q < 7; ++q) s_st[q] = 0;
    // per-phase wall time seen by thread 0 (diagnostic)
    unsigned long long tm_ph[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
    unsigned long long tclk = 0;
    int tick_on = 1;  // DBC_TRACE_SLOT: time one root only
    int own_blk = 0;  // blocks of a published pass the owner ran itself (trace)
    // event trace of the traced slot: code = kind << 56 | level << 32 | items
    auto trace = [&](int kind, int lev, int items) {
        if (kPhaseTimers && tid == 0 && tick_on && a.trace_slot >= 0) {
            unsigned long long t;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            const unsigned long long q = atomicAdd(a.stats + kStTraceN, 1ull);
            if (q < (unsigned long long)kTraceCap) {
                a.stats[kStTrace0 + 2 * q] = ((unsigned long long)kind << 56) |
                                             ((unsigned long long)(lev & 0xFFFFFF) << 32) | (uint32_t)items;
                a.stats[kStTrace0 + 2 * q + 1] = t;
            }
        }
    };
    auto tick = [&](int ph) {
        if (kPhaseTimers && tid == 0 && tick_on) {
            unsigned long long t;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            if (ph >= 0) tm_ph[ph] += t - tclk;
            tclk = t;
        }
    };

    // One help step: scan the board, claim one block of an open request of
    // another worker and run it.  Idle workers (out of roots) loop on it; busy
    // workers call it at their own level boundaries (only there: the block
    // reuses S, I, Bq and s_nbig, which are free between levels).  (cur_owner,
    // cur_seq) caches the chunk loaded into I -- valid only while this CTA runs
    // nothing else.  Returns -2 when every root chain is done (idle), -1 when
    // no block was taken, 1 after running one.
    // one block of a helped down level (owner or helper): short rows in-lane;
    // long rows staged in shared memory (I.v is free outside the up phase) and
    // appended to the owner's queue oBq with one reservation per block
    // (gb[0] rows, gb[1] their entries)
    auto down_block = [&](const DownCtx &c, int i0, int i1, int32_t *oBq, int *gb) {
        if (tid == 0) {
            s_stg[0] = 0;
            s_stg[1] = 0;
        }
        __syncthreads();
        dc_small(c, i0, i1,
                 [&](int i, int len) {
                     const int q = atomicAdd(&s_stg[0], 1);
                     if (q < kChunk)
                         I.v[q] = i;
                     else
                         oBq[atomicAdd(gb, 1)] = i;
                     atomicAdd(&s_stg[1], len);
                 },
                 st_bytes, sc_down);
        __syncthreads();
        const int m = min(s_stg[0], kChunk);
        if (tid == 0) {
            s_stg[2] = m ? atomicAdd(gb, m) : 0;
            if (s_stg[1]) atomicAdd(gb + 1, s_stg[1]);
        }
        __syncthreads();
        for (int i = tid; i < m; i += kBlock) oBq[s_stg[2] + i] = I.v[i];
        __syncthreads();
    };
    auto help_step = [&](bool idle, int &cur_owner, int &cur_seq) -> int {
        // the whole CTA scans the board (one word per thread), first open one wins
        // Priority: the request with the most blocks left (the widest pass of the
        // slowest chain); busy workers only take passes of >= busy_min blocks.
        const int nw = a.help.nworkers;
        if (tid == 0) s_hpick = 0;
        __syncthreads();
        for (int i = tid; i < nw; i += kBlock) {
            const int o = (wk + 1 + i) % nw;
            const unsigned long long w = __ldcg(a.help.word + o);
            const int left = help_nblocks(w) - help_next(w);
            if (help_open(w) && left > 0 && (idle || help_nblocks(w) >= a.busy_min))
                atomicMax((unsigned *)&s_hpick, ((unsigned)min(left, 0xFFFFF) << 12) | (unsigned)i);
        }
        __syncthreads();
        if (tid == 0) {
            int pick = -1, b = -1, sq = -1;
            if (idle && atomicAdd(a.help.roots_left, 0) <= 0) {
                pick = -2;
            } else {
                if (s_hpick != 0) pick = (wk + 1 + (s_hpick & 0xFFF)) % nw;
                if (pick >= 0) {
                    const unsigned long long w = atomicAdd(a.help.word + pick, 1ull << 16);
                    if (help_open(w) && help_next(w) < help_nblocks(w)) {
                        b = help_next(w);
                        sq = help_seq(w);
                    }
                }
            }
            s_hpick = pick;
            s_hb = b;
            s_hseq = sq;
        }
        __syncthreads();
        const int pick = s_hpick, b = s_hb, sq = s_hseq;
        __syncthreads();
        if (pick == -2) return -2;
        if (b < 0) return -1;
        if (pick != cur_owner || sq != cur_seq) {  // a new request: load its chunk
            if (tid == 0) {
                const HelpCtx *src = a.help.ctx + pick;
                s_hctx.root_slot = __ldcg(&src->root_slot);
                s_hctx.l = __ldcg(&src->l);
                s_hctx.g0 = __ldcg(&src->g0);
                s_hctx.lim = __ldcg(&src->lim);
                s_hctx.cnt = __ldcg(&src->cnt);
                s_hctx.nblocks = __ldcg(&src->nblocks);
                s_hctx.E2 = __ldcg(&src->E2);
                s_hctx.E = __ldcg(&src->E);
                s_hctx.kind = __ldcg(&src->kind);
                s_hctx.lb = __ldcg(&src->lb);
                s_hctx.mvalid = __ldcg(&src->mvalid);
                s_hctx.aux = __ldcg(&src->aux);
                __threadfence();  // acquire: drop stale L1 lines of the owner's state
            }
            __syncthreads();
            const ChunkSmem *mir = a.help.mir + pick;
            const int cnt = (s_hctx.kind == 0 || s_hctx.kind == 2) ? s_hctx.cnt : 0;  // kinds 0 and 2 publish a chunk
            if ((s_hctx.kind == 1 || s_hctx.kind == 4 || s_hctx.kind == 5) && s_hctx.mvalid && tid < 32) {  // the root's row (mask bits)
                const int2 rs = row_of(g, a.roots[s_hctx.root_slot], s_hctx.lim);
                const int ds = rs.y - rs.x;
                if (tid < ds && ds <= kMaskDeg) s_hadjs[tid] = ldg_i(g.col + rs.x + tid);
                if (tid == 0) s_hds = ds;
            }
            for (int t = tid; t < cnt; t += kBlock) {
                I.v[t] = __ldcg(&mir->v[t]);
                I.meta[t] = __ldcg(&mir->meta[t]);
                I.beg[t] = __ldcg(&mir->beg[t]);
                I.off[t + 1] = __ldcg(&mir->off[t + 1]);
                I.acc[t] = __ldcg(&mir->acc[t]);
                I.c0[t] = __ldcg(&mir->c0[t]);
                I.c1[t] = __ldcg(&mir->c1[t]);
                I.c2[t] = __ldcg(&mir->c2[t]);
            }
            if (tid == 0) I.off[0] = 0;
            __syncthreads();
            cur_owner = pick;
            cur_seq = sq;
        }
        const HelpCtx cx = s_hctx;
        const Root ost{a.d + (size_t)cx.root_slot * n, a.sd + (size_t)cx.root_slot * n};
        if (cx.kind == 1 || cx.kind == 4) {  // a block of a published down-phase level / its long rows
            DownCtx hd;
            hd.g = g;
            hd.st = ost;
            hd.mark = a.ws.mark + (size_t)pick * n;
            hd.lowrec = a.ws.lowrec + (size_t)pick * n;
            hd.Dv = a.ws.Dv + (size_t)pick * n;
            hd.Dold = a.ws.Dold + (size_t)pick * n;
            hd.Dsig = a.ws.Dsig + (size_t)pick * n;
            hd.mask = a.l2mask + (size_t)cx.root_slot * n;
            hd.err = a.err;
            hd.dcnt = a.help.gapp + pick;
            hd.lowflag = a.help.low + pick;
            hd.adjs = s_hadjs;
            hd.dsr = s_hds;
            hd.L = cx.l;
            hd.lb = cx.lb;
            hd.lim = cx.lim;
            hd.mvalid = cx.mvalid;
            hd.del = a.del;
            hd.epoch = cx.E >> 2;
            hd.mD = cx.E | kDown;
            int32_t *oBq = a.ws.Bq + (size_t)pick * n;  // the owner's long-row queue
            if (cx.kind == 1) {
                const int kDownBlock = a.hd_block;
                int *gb = a.help.gbig + 2 * pick;
                down_block(hd, b * kDownBlock, min(cx.cnt, (b + 1) * kDownBlock), oBq, gb);
            } else {
                dl_block<true>(hd, S, oBq, a.ws.U1 + (size_t)pick * n, cx.cnt, b * kDlEntries,
                               min(cx.E2, (b + 1) * kDlEntries), a.ws.dacc + (size_t)pick * n, &s_t0, st_bytes,
                               sc_down);
            }
        } else if (cx.kind == 5) {  // a block of a published in-lane up-level pass
            UpCtx uc;
            uc.g = g;
            uc.st = ost;
            uc.mark = a.ws.mark + (size_t)pick * n;
            uc.dacc = a.ws.dacc + (size_t)pick * n;
            uc.bc = a.bc;
            uc.mask = a.l2mask + (size_t)cx.root_slot * n;
            uc.Dv = a.ws.Dv + (size_t)pick * n;
            uc.Dold = a.ws.Dold + (size_t)pick * n;
            uc.Rv = a.ws.Rv + (size_t)pick * n;
            uc.Rl = a.ws.Rl + (size_t)pick * n;
            uc.Ul = a.ws.Bq + (size_t)pick * n;
            uc.Uo = ((cx.aux >> 30) & 1 ? a.ws.U1 : a.ws.U0) + (size_t)pick * n;
            uc.Dsig = a.ws.Dsig + (size_t)pick * n;
            uc.adjs = s_hadjs;
            uc.gU = a.help.gU + (size_t)pick * n;
            uc.gapp = a.help.gapp + pick;
            uc.xcnt = a.help.gbig + 2 * pick;
            uc.X = a.ws.X + (size_t)pick * kXcap;
            uc.l = cx.l;
            uc.b0 = cx.lb;
            uc.nDl = cx.E2;
            uc.ucnt = cx.aux & ((1 << 30) - 1);
            uc.g0 = cx.g0;
            uc.lim = cx.lim;
            uc.mok = cx.mvalid;
            uc.E = cx.E;
            uc.mU = cx.E | kUp;
            uc.mD = cx.E | kDown;
            up_block(uc, b * a.hd_block, min(cx.cnt, (b + 1) * a.hd_block), st_bytes, sc_up3);
        } else if (cx.kind == 3) {  // a block of a published removal pass (Case 3)
            RemCtx hr;
            hr.g = g;
            hr.st = ost;
            hr.mark = a.ws.mark + (size_t)pick * n;
            hr.dacc = a.ws.dacc + (size_t)pick * n;
            hr.Dv = a.ws.Dv + (size_t)pick * n;
            hr.Dold = a.ws.Dold + (size_t)pick * n;
            hr.Dsig = a.ws.Dsig + (size_t)pick * n;
            hr.Rv = a.ws.Rv + (size_t)pick * n;
            hr.Rl = a.ws.Rl + (size_t)pick * n;
            hr.rcnt = a.help.gapp + pick;
            hr.rmax = a.help.low + pick;
            hr.g0 = cx.g0;
            hr.lim = cx.lim;
            hr.E = cx.E;
            hr.mD = cx.E | kDown;
            hr.mU = cx.E | kUp;
            const int kRemBlock = a.hd_block;
            rem_range(hr, S, s_l1, a.ws.Bq + (size_t)wk * n, &s_nbig, b * kRemBlock,
                      min(cx.cnt, (b + 1) * kRemBlock), st_bytes, sc_rem);
        } else if (cx.kind == 2) {  // a block of a published delta-pull pass (C1)
            const int e0 = b * a.he_entries, e1 = min(cx.E2, (b + 1) * a.he_entries);
            for (int t = tid; t < cx.cnt; t += kBlock) I.acc[t] = 0.0;
            __syncthreads();
            auto colf = [&](int t, int e) { return ldg_i(g.col + I.beg[t] + e - I.off[t]); };
            flat_entries<true>(I.off, cx.cnt, e1, colf, ost, nullptr, [&](int dy) { return dy == cx.l + 1; },
                               I.acc, [&](int t, int, int dy, double2 q, uint32_t) -> double {
                                   st_bytes += 8;
                                   if (dy != cx.l + 1) return 0.0;
                                   return __dmul_rn(__ddiv_rn(I.c0[t], q.x), __dadd_rn(1.0, q.y));
                               }, e0);
            ChunkSmem *mir = a.help.mir + pick;
            for (int t = tid; t < cx.cnt; t += kBlock)
                if (I.acc[t] != 0.0) atomicAdd(&mir->acc[t], I.acc[t]);
        } else {
            help_run_block<true>(I, b * a.he_entries, min(cx.E2, (b + 1) * a.he_entries), g, ost,
                                 a.ws.mark + (size_t)pick * n, a.ws.dacc + (size_t)pick * n,
                                 a.help.gU + (size_t)pick * n, a.help.gapp + pick, cx, st_bytes);
        }
        __syncthreads();
        if (tid == 0) {  // release by one thread after the CTA barrier
            __threadfence();
            atomicAdd(a.help.done + pick, 1);
            atomicAdd(stat_lane(a.stats) + kStHelpBlk, 1ull);
        }
        return 1;
    };
    // a busy worker at a level boundary: take up to a.busy_help blocks of other
    // workers' open requests (the heavy chains' wide levels do not wait for
    // idle workers).  s_hopen was sampled during the previous level; every
    // thread reads the same value (written before a barrier).
    auto busy_help = [&]() {
        if (!a.help.word || a.busy_help <= 0 || (s_hopen & 0xFFFF) == 0) return;
        int co = -1, cs = -1;
        for (int q = 0; q < a.busy_help; ++q) {
            if (help_step(false, co, cs) < 0) break;
            if (tid == 0) atomicAdd(stat_lane(a.stats) + kStBusyBlk, 1ull);
        }
    };
    // sampled at a level start by thread 0, published at the level end:
    // open wide requests (busy workers help) and idle workers (a pass is worth
    // publishing only if someone can take its blocks)
    auto sample_open = [&]() {
        return (tid == 0 && a.help.word)
                   ? min(__ldcg(a.help.roots_left + 1), 0xFFFF) | (min(__ldcg(a.help.roots_left + 2), 0x7FFF) << 16)
                   : 0;
    };
    // publish a pass of nb blocks?  (idle helpers exist, or busy ones take passes this wide)
    auto worth = [&](int nb) { return (s_hopen >> 16) > 0 || (a.busy_help > 0 && nb >= a.busy_min); };


    if (tid == 0) {
        s_nbig = 0;
        s_nbigI = 0;
        s_nl1 = 0;
        s_noext = 0;
        s_hopen = 0;
        s_nx[0] = 0;
        s_nx[1] = 0;
    }

    for (;;) {
        if (tid == 0) {
            const int q = atomicAdd(a.next_slot, 1);
            const int cnt = a.slot_list ? a.slot_count : a.k_loc;
            s_slot = q < cnt ? (a.slot_list ? a.slot_list[q] : q) : -1;
            if (s_slot < 0 && a.steal_list) {  // the other lane's roots: no lane waits on the other's residency
                const int q2 = atomicAdd(a.steal_next, 1);
                s_slot = q2 < a.steal_count ? a.steal_list[q2] : -1;
            }
        }
        __syncthreads();
        const int slot = s_slot;
        __syncthreads();
        if (slot < 0) break;
        const Root st{a.d + (size_t)slot * n, a.sd + (size_t)slot * n};
        const int sroot = a.roots[slot];
        tick_on = a.trace_slot < 0 || a.trace_slot == slot;
        uint32_t *mask = a.l2mask + (size_t)slot * n;
        if (a.root_prof && tid == 0) {
            unsigned long long t;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            s_prof[0] = t;
            s_prof[1] = 0;
            s_prof[2] = s_st[0];
            s_prof[3] = (unsigned long long)sc_down + sc_rem + sc_dpull + sc_dpush + sc_up2 + sc_up3;
            s_prof[4] = s_st[5] + s_st[6];
        }

        // Insertions are taken in windows (ws.wcap of them, or 1 with
        // DBC_FLAG_NO_MERGE).  A window is ONE job (R18): every
        // insertion e = (a, b) with d[a] < d[b] at the window start is a seed
        // of level d[a] + 1, injected when the down phase reaches that level if
        // a still has that distance (else a was lowered, is in D, and its own
        // row walk covers e); b is then lowered (Case 3) or just
        // claimed (Case 2).  The result is the state of the graph
        // with all of the window's edges -- what the insertions one by one give.
        const int win = a.merge ? a.ws.wcap : 1;
        int ins = a.ins_begin;
        while (ins < a.ins_end) {
            const int wend = min(ins + win, a.ins_end);
            const int nwin = wend - ins;
            if (tid == 0) {
                s_job[2] = INT32_MAX;  // lowest seed level
                s_job[7] = 0;          // deepest seed level
                s_job[3] = 0;          // any distance lowered in this job
                s_wcnt[0] = 0;
                s_wcnt[1] = 0;
            }
            __syncthreads();
            {  // classification (K2) against the window-start distances
                int lmin = INT32_MAX, lmax = 0, cw = 0, c3n = 0;
                for (int q = tid; q < nwin; q += kBlock) {
                    const int u = __ldg(a.ins_u + ins + q), v = __ldg(a.ins_v + ins + q);
                    const int du = st.dist(u), dv = st.dist(v);
                    const bool work = du != dv;
                    const int lev = work ? min(du, dv) + 1 : INT32_MAX;
                    Wul[q] = du < dv ? v : u;
                    Wlev[q] = lev;
                    if (work) {
                        ++cw;
                        c3n += min(du, dv) + 1 != max(du, dv);
                        lmin = min(lmin, lev);
                        lmax = max(lmax, lev);
                    }
                }
                // warp-aggregated, then one shared atomic per warp
#pragma unroll
                for (int o = 16; o; o >>= 1) {
                    cw += __shfl_xor_sync(kFull, cw, o);
                    c3n += __shfl_xor_sync(kFull, c3n, o);
                    lmin = min(lmin, __shfl_xor_sync(kFull, lmin, o));
                    lmax = max(lmax, __shfl_xor_sync(kFull, lmax, o));
                }
                if ((tid & 31) == 0 && cw) {
                    atomicAdd(&s_wcnt[0], cw);
                    atomicAdd(&s_wcnt[1], c3n);
                    atomicMin(&s_job[2], lmin);
                    atomicMax(&s_job[7], lmax);
                }
            }
            __syncthreads();
            {
                const int nw = s_wcnt[0], n3 = s_wcnt[1];
                if (tid == 0) {
                    s_st[2] += nwin - nw;
                    s_st[3] += nw - n3;
                    s_st[4] += n3;
                    st_bytes += 8ull * nwin;
                    if (nw > 1) {
                        atomicAdd(stat_lane(a.stats) + kStGroups, 1ull);
                        atomicAdd(stat_lane(a.stats) + kStGroupIns, (unsigned long long)nw);
                    }
                }
                if (nw == 0) {  // Case 1 throughout: nothing changes
                    if (a.scen && tid == 0) a.scen[(size_t)ins * a.k_loc + slot] = 1;
                    ins = wend;
                    __syncthreads();  // the counters are reset by the next window
                    continue;
                }
            }
            {
                if (a.del) ++epoch;  // deletion: one epoch for the affected-set search, one for the job
                ++epoch;
                if (tid == 0) ++s_prof[1];
                if (tid == 0) s_touch0 = s_st[0];  // scenario log (thread 0's counter)
                const uint32_t E = epoch << 2;
                const uint32_t mD = E | kDown, mU = E | kUp;
                // the job's insertions and the graph as of lim; a deletion sees
                // every entry (tombstoned edge excluded) and has no new edge
                const int g0 = a.del ? INT32_MAX : ins, lim = a.del ? INT32_MAX - 1 : wend - 1;
                if (tid < 32) {  // warp 0: the root's row as of this job (level-2 masks)
                    const int2 rs = row_of(g, sroot, lim);
                    const int dsr = rs.y - rs.x;
                    if (dsr <= kMaskDeg && tid < dsr) s_adjs[tid] = ldg_i(g.col + rs.x + tid);
                    if (tid == 0) {
                        const int built = a.mask_ds[slot];
                        // 1: masks valid; 2: the root gained a neighbour -> rebuild after the down phase
                        s_job[4] = (dsr > kMaskDeg) ? 0 : (built == dsr ? 1 : 2);
                        s_job[5] = dsr;
                        if (dsr > kMaskDeg && built >= 0) a.mask_ds[slot] = -1;
                    }
                }
                if (tid == 0) {
                    Doff[0] = 0;
                    s_dcnt = 0;
                    s_ucnt2[0] = 0;
                    s_ucnt2[1] = 0;
                    s_rcnt = 0;
                    s_rmax = 0;
                }
                __syncthreads();
                if (a.del) {
                    // ---- edge deletion (decremental update, R20) ----
                    // The edge (u_high, u_low) is already a tombstone in both rows.
                    if (tid == 0) {
                        const int u = __ldg(a.ins_u + ins), v = __ldg(a.ins_v + ins);
                        const int uh = st.d[u] < st.d[v] ? u : v, ul = uh == u ? v : u;
                        s_del[0] = uh;
                        s_del[1] = ul;
                        s_del[2] = 0;
                        s_del[3] = 0;
                        s_del[4] = 0;
                        s_del[5] = 0;
                        const double2 q = st.sd[ul];
                        s_delsd[0] = q.x;
                        s_delsd[1] = q.y;
                    }
                    __syncthreads();
                    const int ul = s_del[1];
                    const int Lul = st.d[ul];
                    if (tid < 32) {  // does u_low keep a predecessor?
                        const int2 r = row_of(g, ul, lim);
                        bool keep = false;
                        for (int j = r.x + tid; j < r.y && !keep; j += 32) keep = st.d[ldg_i(g.col + j)] == Lul - 1;
                        if (__any_sync(kFull, keep) && tid == 0) s_del[5] = 1;
                    }
                    __syncthreads();
                    if (s_del[5]) {  // distances unchanged: sigma shrinks below u_low (seed u_low)
                        if (tid == 0) {
                            Rv[0] = ul;
                            Rl[0] = Lul;
                            s_del[3] = 1;
                            s_job[2] = Lul;
                            s_job[7] = Lul;
                        }
                    } else {
                        // A = the vertices whose distance grows: u_low, then level by level
                        // every old successor all of whose predecessors are in A.  A is
                        // raised to INF (old d kept in lowrec, tagged with the job epoch);
                        // successors that keep a predecessor lose paths: seeds at their level.
                        const uint32_t mA = ((epoch - 1) << 2) | kDown;  // search epoch
                        if (tid == 0) {
                            lowrec[ul] = ((unsigned long long)epoch << 32) | (uint32_t)Lul;
                            st.d[ul] = kInf;
                            Ua[0] = ul;
                            s_del[2] = 1;
                            s_job[3] = 1;
                            s_wcnt[1] = 1;  // a distance changes: reported as Case 3
                            --s_st[3];
                            ++s_st[4];
                        }
                        __syncthreads();
                        int fb = 0, fe = 1, la = Lul;
                        while (fb < fe) {
                            for (int i = fb + tid; i < fe; i += kBlock) {
                                const int x = Ua[i];
                                const int2 r = row_of(g, x, lim);
                                for (int j = r.x; j < r.y; ++j) {
                                    const int y = ldg_i(g.col + j);
                                    if (st.d[y] == la + 1 && atomicMax(mark + y, mA) < mA)
                                        Bq[atomicAdd(&s_del[4], 1)] = y;
                                }
                            }
                            __syncthreads();
                            const int nc = s_del[4];
                            for (int i = tid; i < nc; i += kBlock) {
                                const int y = Bq[i];
                                const int2 r = row_of(g, y, lim);
                                bool keep = false;
                                for (int j = r.x; j < r.y && !keep; ++j) keep = st.d[ldg_i(g.col + j)] == la;
                                if (keep) {  // y keeps its level, its sigma changes
                                    const int q = atomicAdd(&s_del[3], 1);
                                    Rv[q] = y;
                                    Rl[q] = la + 1;
                                } else {
                                    lowrec[y] = ((unsigned long long)epoch << 32) | (uint32_t)(la + 1);
                                    Ua[atomicAdd(&s_del[2], 1)] = y;
                                }
                            }
                            __syncthreads();
                            for (int i = tid; i < nc; i += kBlock) {  // raise the new A level (after every check)
                                const int y = Bq[i];
                                if ((uint32_t)(lowrec[y] >> 32) == epoch) st.d[y] = kInf;
                            }
                            if (tid == 0) s_del[4] = 0;
                            __syncthreads();
                            fb = fe;
                            fe = s_del[2];
                            ++la;
                        }
                        // seeds of A: one more than the nearest vertex outside A
                        const int na = s_del[2];
                        for (int i = tid; i < na; i += kBlock) {
                            const int x = Ua[i];
                            const int2 r = row_of(g, x, lim);
                            int t = kInf;
                            for (int j = r.x; j < r.y; ++j) {
                                const int dy = st.d[ldg_i(g.col + j)];
                                if (dy != kInf) t = min(t, dy + 1);
                            }
                            if (t != kInf) {
                                const int q = atomicAdd(&s_del[3], 1);
                                Rv[q] = x;
                                Rl[q] = t;
                            }
                        }
                        __syncthreads();
                        const int ns = s_del[3];
                        int lmin = INT32_MAX, lmax = 0;
                        for (int i = tid; i < ns; i += kBlock) {
                            lmin = min(lmin, Rl[i]);
                            lmax = max(lmax, Rl[i]);
                        }
#pragma unroll
                        for (int o = 16; o; o >>= 1) {
                            lmin = min(lmin, __shfl_xor_sync(kFull, lmin, o));
                            lmax = max(lmax, __shfl_xor_sync(kFull, lmax, o));
                        }
                        if (tid == 0) {
                            s_job[2] = INT32_MAX;
                            s_job[7] = 0;
                        }
                        __syncthreads();
                        if ((tid & 31) == 0) {
                            atomicMin(&s_job[2], lmin);
                            atomicMax(&s_job[7], lmax);
                        }
                        __syncthreads();
                        if (tid == 0 && ns == 0) {  // everything below u_low is cut off
                            s_job[2] = 1;
                            s_job[7] = 1;
                        }
                    }
                    __syncthreads();
                }
                const int L0 = s_job[2];
                const int Lseed = s_job[7];
                const int mstate = s_job[4], dsr = s_job[5];
                // enqueue the seeds of level Lq (between levels: no concurrent lowering)
                auto inject = [&](int Lq) {
                    if (a.del) {  // deletion seeds (u_low, or A / lost-path vertices)
                        const int ns = s_del[3];
                        for (int q = tid; q < ns; q += kBlock) {
                            if (Rl[q] != Lq) continue;
                            const int b = Rv[q];
                            const int db = st.d[b];
                            if (db < Lq) continue;  // reached earlier by the search
                            if (db > Lq) atomicMin(st.d + b, Lq);  // raised vertex: old d already recorded
                            if (atomicMax(mark + b, mD) < mD) Dv[atomicAdd(&s_dcnt, 1)] = b;
                        }
                        return;
                    }
                    for (int q = tid; q < nwin; q += kBlock) {
                        if (Wlev[q] != Lq) continue;
                        const int b = Wul[q];
                        const int u = __ldg(a.ins_u + ins + q), v = __ldg(a.ins_v + ins + q);
                        const int hi = (u == b) ? v : u;
                        if (st.d[hi] != Lq - 1) continue;  // lowered: in D, its row walk covers e
                        const int db = st.d[b];
                        if (db < Lq) continue;
                        if (db > Lq) {  // Case 3: pull b up to level Lq
                            const int old = atomicMin(st.d + b, Lq);
                            if (old > Lq) {
                                lowrec[b] = ((unsigned long long)epoch << 32) | (uint32_t)old;
                                s_job[3] = 1;
                            }
                        }
                        if (atomicMax(mark + b, mD) < mD) Dv[atomicAdd(&s_dcnt, 1)] = b;
                    }
                };
                inject(L0);
                __syncthreads();
                const int le0 = s_dcnt;
                if (tid == 0) Doff[1] = le0;
                const bool mvalid = mstate == 1;  // masks usable during this job's down phase

                tick(-1);
                // ================= down phase (K3) =================
                int L = L0, lb = 0, le = le0, nlev = 1;
                DownCtx dc;
                dc.g = g;
                dc.st = st;
                dc.mark = mark;
                dc.lowrec = lowrec;
                dc.Dv = Dv;
                dc.Dold = Dold;
                dc.Dsig = Dsig;
                dc.mask = mask;
                dc.err = a.err;
                dc.dcnt = &s_dcnt;
                dc.lowflag = &s_job[3];
                dc.adjs = s_adjs;
                dc.dsr = dsr;
                dc.lim = lim;
                dc.mvalid = mvalid;
                dc.del = a.del;
                dc.epoch = epoch;
                dc.mD = mD;
                while (true) {
#ifndef DBC_NO_BUSY_SITES
                    busy_help();
#endif
                    const int hopen_pf = sample_open();
                    trace(1, L, le - lb);
                    dc.L = L;
                    dc.lb = lb;
                    const int items = le - lb;
                    const int kDownBlock = a.hd_block;
                    DownCtx gd = dc;  // appends and the lowering flag through global memory (helped passes)
                    gd.dcnt = a.help.gapp + wk;
                    gd.lowflag = a.help.low + wk;
                    int nrows = 0, nent = 0;  // the level's long rows (queued in Bq) and their entries
                    if (a.help.word && items >= a.hd_min && worth((items + kDownBlock - 1) / kDownBlock)) {
                        // a wide level: published, idle workers take blocks of items; their
                        // long rows are queued in this worker's Bq for the entry-balanced pass
                        const int nblk = (items + kDownBlock - 1) / kDownBlock;
                        if (tid == 0) {
                            HelpCtx cx;
                            cx.root_slot = slot;
                            cx.l = L;
                            cx.g0 = g0;
                            cx.lim = lim;
                            cx.cnt = items;
                            cx.nblocks = nblk;
                            cx.E2 = 0;
                            cx.E = E;
                            cx.kind = 1;
                            cx.lb = lb;
                            cx.mvalid = mvalid;
                            a.help.ctx[wk] = cx;
                            a.help.done[wk] = 0;
                            a.help.gapp[wk] = s_dcnt;
                            a.help.low[wk] = 0;
                            a.help.gbig[2 * wk] = 0;
                            a.help.gbig[2 * wk + 1] = 0;
                            __threadfence();
                            atomicAdd(stat_lane(a.stats) + kStHelpReq, 1ull);
                            atomicAdd(stat_lane(a.stats) + kStHelpBlkAll, (unsigned long long)nblk);
                            hseq = (hseq + 1) & 0xFFFF;
                            atomicExch(a.help.word + wk, help_pack(1, nblk, 0, hseq));
                            if (nblk >= a.busy_min) atomicAdd(a.help.roots_left + 1, 1);  // open wide requests
                        }
                        int *gb = a.help.gbig + 2 * wk;
                        for (;;) {  // the owner takes blocks too
                            if (tid == 0) {
                                const unsigned long long w = atomicAdd(a.help.word + wk, 1ull << 16);
                                s_hb = help_next(w) < nblk ? help_next(w) : -1;
                            }
                            __syncthreads();
                            const int b = s_hb;
                            __syncthreads();
                            if (b < 0) break;
                            ++own_blk;
                            down_block(gd, b * kDownBlock, min(items, (b + 1) * kDownBlock), Bq, gb);
                            if (tid == 0) {
                                __threadfence();
                                atomicAdd(a.help.done + wk, 1);
                            }
                        }
                        trace(6, 1, own_blk | (nblk << 16));
                        own_blk = 0;
                        if (tid == 0) {  // wait for the helpers' blocks, then close
                            while (atomicAdd(a.help.done + wk, 0) < nblk) __nanosleep(256);
                            atomicExch(a.help.word + wk, help_pack(0, 0, 0, hseq));
                            if (nblk >= a.busy_min) atomicSub(a.help.roots_left + 1, 1);
                            __threadfence();
                            s_dcnt = __ldcg(a.help.gapp + wk);
                            if (__ldcg(a.help.low + wk)) s_job[3] = 1;
                            s_nbig = __ldcg(gb);
                            s_nent = __ldcg(gb + 1);
                        }
                        __syncthreads();
                    } else {
                        if (tid == 0) s_nent = 0;
                        __syncthreads();
                        dc_small(dc, 0, items,
                                 [&](int i, int len) {
                                     Bq[atomicAdd(&s_nbig, 1)] = i;
                                     atomicAdd(&s_nent, len);
                                 },
                                 st_bytes, sc_down);
                        __syncthreads();
                    }
                    nrows = s_nbig;
                    nent = s_nent;
                    if (a.help.word && nent >= a.dl_min && worth(nent / kDlEntries)) {
                        // long rows with many entries (hub neighbourhoods): entry-balanced
                        // blocks, owner and helpers; per-row results completed by the owner
                        int32_t *Boff = Ub;  // free during the down phase
                        const int tot = dl_offsets(dc, Bq, Boff, nrows, I.off, &s_tot);
                        const int nblk = (tot + kDlEntries - 1) / kDlEntries;
                        trace(9, nrows, tot);
                        if (tid == 0) {
                            HelpCtx cx;
                            cx.root_slot = slot;
                            cx.l = L;
                            cx.g0 = g0;
                            cx.lim = lim;
                            cx.cnt = nrows;
                            cx.nblocks = nblk;
                            cx.E2 = tot;
                            cx.E = E;
                            cx.kind = 4;
                            cx.lb = lb;
                            cx.mvalid = mvalid;
                            a.help.ctx[wk] = cx;
                            a.help.done[wk] = 0;
                            a.help.gapp[wk] = s_dcnt;
                            a.help.low[wk] = 0;
                            __threadfence();
                            atomicAdd(stat_lane(a.stats) + kStHelpReq, 1ull);
                            atomicAdd(stat_lane(a.stats) + kStHelpBlkAll, (unsigned long long)nblk);
                            hseq = (hseq + 1) & 0xFFFF;
                            atomicExch(a.help.word + wk, help_pack(1, nblk, 0, hseq));
                            if (nblk >= a.busy_min) atomicAdd(a.help.roots_left + 1, 1);
                        }
                        for (;;) {  // the owner takes blocks too
                            if (tid == 0) {
                                const unsigned long long w = atomicAdd(a.help.word + wk, 1ull << 16);
                                s_hb = help_next(w) < nblk ? help_next(w) : -1;
                            }
                            __syncthreads();
                            const int b = s_hb;
                            __syncthreads();
                            if (b < 0) break;
                            ++own_blk;
                            dl_block<false>(gd, S, Bq, Boff, nrows, b * kDlEntries, min(tot, (b + 1) * kDlEntries),
                                            dacc, &s_t0, st_bytes, sc_down);  // ends with a barrier
                            if (tid == 0) {
                                __threadfence();
                                atomicAdd(a.help.done + wk, 1);
                            }
                        }
                        trace(6, 4, own_blk | (nblk << 16));
                        own_blk = 0;
                        if (tid == 0) {  // wait for the helpers' blocks, then close
                            while (atomicAdd(a.help.done + wk, 0) < nblk) __nanosleep(256);
                            atomicExch(a.help.word + wk, help_pack(0, 0, 0, hseq));
                            if (nblk >= a.busy_min) atomicSub(a.help.roots_left + 1, 1);
                            __threadfence();
                            s_dcnt = __ldcg(a.help.gapp + wk);
                            if (__ldcg(a.help.low + wk)) s_job[3] = 1;
                        }
                        __syncthreads();
                        dl_finish(dc, Bq, nrows, dacc, st_bytes);  // ends with a barrier
                    } else if (nrows > 0) {
                        dc_big(dc, S, Bq, nrows, st_bytes, sc_down);
                    }
                    if (L < Lseed) {  // seeds of the next level (claimed children stay once)
                        inject(L + 1);
                        __syncthreads();
                    }
                    const int ne = s_dcnt;
                    __syncthreads();  // everyone has read nbig / ne
                    if (tid == 0) {
                        s_nbig = 0;
                        s_hopen = hopen_pf;
                        if (ne != le || L < Lseed) Doff[nlev + 1] = ne;
                    }
                    __syncthreads();  // reset visible before the next level enqueues
                    if (ne == le && L >= Lseed) break;
                    lb = le;
                    le = ne;
                    ++nlev;
                    ++L;
                }
                // D levels: level L0 + j occupies Dv[Doff[j] .. Doff[j+1]), j < nlev
                const int LmaxD = L0 + nlev - 1;
                const int dtotal = le;
                if (tid == 0) s_st[5] += nlev;
                if (tid == 0) {
                    s_st[1] += dtotal;
                    s_st[0] += dtotal;
                }

                // the root gained a neighbour (Case 3 with u_high = root): rebuild its masks
                if (mstate == 2) {
                    build_l2masks(g, st, mask, row_of(g, sroot, lim), lim);
                    if (tid == 0) a.mask_ds[slot] = dsr;
                }
                const bool mok = mstate != 0;  // masks valid for the up phase
                const bool case3 = s_job[3] != 0;  // some distance was lowered (read after the level barriers)

                if (a.del) {
                    // deletion: A vertices the search never reached are cut off from
                    // the root (d = INF, sigma = delta = 0, P:150-159 reading R4); the
                    // deleted edge carried u_low's old contribution to u_high
                    const int na = s_del[2];
                    for (int i = tid; i < na; i += kBlock) {
                        const int x = Ua[i];
                        if (st.d[x] != kInf) continue;
                        const double od = st.sd[x].y;
                        if (od != 0.0) atomicAdd(a.bc + x, -od);
                        st.sd[x] = make_double2(0.0, 0.0);
                        st_bytes += 32;
                    }
                    if (tid == 0) {
                        const int uh = s_del[0];
                        const int dh = st.d[uh];
                        if (dh >= 1) {  // the root's delta is never used
                            atomicAdd(dacc + uh, -__ddiv_rn(1.0 + s_delsd[1], s_delsd[0]));
                            if (atomicMax(mark + uh, mU) < E) {
                                const int pos = atomicAdd(&s_rcnt, 1);
                                Rv[pos] = uh;
                                Rl[pos] = dh;
                                atomicMax(&s_rmax, dh);
                            }
                        }
                    }
                    __syncthreads();
                }

                tick(0);
                // ================= (0) Case-3 removal pushes =================
                trace(3, 0, dtotal);
                if (case3) {
                    RemCtx rc;
                    rc.g = g;
                    rc.st = st;
                    rc.mark = mark;
                    rc.dacc = dacc;
                    rc.Dv = Dv;
                    rc.Dold = Dold;
                    rc.Dsig = Dsig;
                    rc.Rv = Rv;
                    rc.Rl = Rl;
                    rc.rcnt = &s_rcnt;
                    rc.rmax = &s_rmax;
                    rc.g0 = g0;
                    rc.lim = lim;
                    rc.E = E;
                    rc.mD = mD;
                    rc.mU = mU;
                    const int kRemBlock = a.hd_block;
                    if (a.help.word && dtotal >= a.hd_min && worth((dtotal + a.hd_block - 1) / a.hd_block)) {
                        // a wide pass: published, idle and busy workers take blocks of D
                        // (appends to R and the deepest target level go through global memory)
                        const int nblk = (dtotal + kRemBlock - 1) / kRemBlock;
                        if (tid == 0) {
                            HelpCtx cx;
                            cx.root_slot = slot;
                            cx.l = 0;
                            cx.g0 = g0;
                            cx.lim = lim;
                            cx.cnt = dtotal;
                            cx.nblocks = nblk;
                            cx.E2 = 0;
                            cx.E = E;
                            cx.kind = 3;
                            cx.lb = 0;
                            cx.mvalid = 0;
                            a.help.ctx[wk] = cx;
                            a.help.done[wk] = 0;
                            a.help.gapp[wk] = s_rcnt;
                            a.help.low[wk] = s_rmax;
                            __threadfence();
                            atomicAdd(stat_lane(a.stats) + kStHelpReq, 1ull);
                            atomicAdd(stat_lane(a.stats) + kStHelpBlkAll, (unsigned long long)nblk);
                            hseq = (hseq + 1) & 0xFFFF;
                            atomicExch(a.help.word + wk, help_pack(1, nblk, 0, hseq));
                            if (nblk >= a.busy_min) atomicAdd(a.help.roots_left + 1, 1);  // open wide requests
                        }
                        RemCtx gr = rc;
                        gr.rcnt = a.help.gapp + wk;
                        gr.rmax = a.help.low + wk;
                        for (;;) {  // the owner takes blocks too
                            if (tid == 0) {
                                const unsigned long long w = atomicAdd(a.help.word + wk, 1ull << 16);
                                s_hb = help_next(w) < nblk ? help_next(w) : -1;
                            }
                            __syncthreads();
                            const int b = s_hb;
                            __syncthreads();
                            if (b < 0) break;
                            ++own_blk;
                            rem_range(gr, S, s_l1, Bq, &s_nbig, b * kRemBlock, min(dtotal, (b + 1) * kRemBlock),
                                      st_bytes, sc_rem);  // ends with a barrier
                            if (tid == 0) {
                                __threadfence();
                                atomicAdd(a.help.done + wk, 1);
                            }
                        }
                        trace(6, 3, own_blk | (nblk << 16));
                        own_blk = 0;
                        if (tid == 0) {  // wait for the helpers' blocks, then close
                            while (atomicAdd(a.help.done + wk, 0) < nblk) __nanosleep(256);
                            atomicExch(a.help.word + wk, help_pack(0, 0, 0, hseq));
                            if (nblk >= a.busy_min) atomicSub(a.help.roots_left + 1, 1);
                            __threadfence();
                            s_rcnt = __ldcg(a.help.gapp + wk);
                            s_rmax = __ldcg(a.help.low + wk);
                        }
                        __syncthreads();
                    } else {
                        rem_range(rc, S, s_l1, Bq, &s_nbig, 0, dtotal, st_bytes, sc_rem);
                    }
                }
                const int rcnt = s_rcnt;
                // a deletion's removal targets can sit one level above the seeds (u_high)
                const int Lstop = a.del ? min(L0, st.d[s_del[0]]) : L0;
                const int Lmax = max(LmaxD, s_rmax);
                if (tid == 0) s_st[0] += rcnt;

                tick(1);
                // ================= up phase (K4 + Alg. 8) =================
                int *Ucur = Ua, *Unext = Ub;  // overflow beyond kUcap entries
                int ucur_sel = 0;
                int ucnt = 0;
                for (int l = Lmax; l >= 1; --l) {
                    if (l < Lstop && ucnt == 0) break;  // nothing left above the insertion
#ifndef DBC_NO_BUSY_SITES
                    busy_help();
#endif
                    const int hopen_pf = sample_open();
                    trace(2, l, ucnt + rcnt + ((l >= L0 && l <= LmaxD) ? Doff[l - L0 + 1] - Doff[l - L0] : 0));
                    const bool push = l >= 2;          // level-1 vertices only feed the root
                    if (tid == 0) ++s_st[6];
                    // queue p for level l-1 unless already queued: the prefetched mark
                    // filters the common case, the returning atomic elects one
                    // appender among concurrent pushers (no duplicates)
                    auto claim_up = [&](int y, uint32_t my) {
                        if (my >= E) return;
                        if (atomicMax(mark + y, mU) >= E) return;
                        const int pos = atomicAdd(&s_ucnt2[ucur_sel ^ 1], 1);
                        if (pos < kUcap)
                            s_un[ucur_sel ^ 1][pos] = y;
                        else
                            Unext[pos - kUcap] = y;
                    };
                    // up vertex x (not in D): push sigma[p]/sigma[x] * Ddelta[x] upwards
                    auto up_visit = [&](double gx, double sx, int pp, double sp, uint32_t mp) {
                        (void)sp;
                        atomicAdd(dacc + pp, __ddiv_rn(gx, sx));
                        st_bytes += 24;
                        claim_up(pp, mp);
                    };
                    auto up_finish = [&](int x, double gx, double odel) {
                        dacc[x] = 0.0;
                        st.sd[x].y = odel + gx;
                        atomicAdd(a.bc + x, gx);
                        st_bytes += 16 + 16;  // delta RMW, BC RMW (40 B per up vertex)
                    };
                    // down vertex x: pull delta (Eq. (2)), then push new-minus-old contributions
                    auto dpull_visit = [&](double sx, int dy, double sy, double dly) -> double {
                        if (dy != l + 1) return 0.0;
                        st_bytes += 16;
                        return __dmul_rn(__ddiv_rn(sx, sy), __dadd_rn(1.0, dly));
                    };
                    auto dpush_visit = [&](int x, double sx, double dn, double odel, double osig,
                                           int meta, int pp, double sp, uint32_t mp) {
                        if (mp == mD) return;
                        (void)sp;
                        double dlt = __ddiv_rn(1.0 + dn, sx);
                        if ((meta & kMetaNotPulled) && !((meta & kMetaNew) && new_edge(g, x, pp, g0, lim)))
                            dlt = __dsub_rn(dlt, __ddiv_rn(1.0 + odel, osig));
                        atomicAdd(dacc + pp, dlt);
                        st_bytes += 24;
                        claim_up(pp, mp);
                    };
                    auto d_finish = [&](int x, double dn, double odel) {
                        st.sd[x].y = dn;
                        atomicAdd(a.bc + x, dn - odel);
                        st_bytes += 8 + 16;  // delta write, BC RMW
                    };

                    int b0 = 0, b1 = 0;
                    if (l >= L0 && l <= LmaxD) {
                        b0 = Doff[l - L0];
                        b1 = Doff[l - L0 + 1];
                    }
                    const int nDl = b1 - b0;
                    if (l == 2) {  // level-1 set = the root's row as of this insertion
                        if (tid == 0) {
                            const int2 rr = row_of(g, sroot, lim);
                            s_ds = (rr.y - rr.x <= kAdjCap) ? rr.y - rr.x : -1;
                        }
                        __syncthreads();
                        if (s_ds > 0) {
                            const int2 rr = row_of(g, sroot, lim);
                            for (int j = tid; j < s_ds; j += kBlock) {
                                const int pj = ldg_i(g.col + rr.x + j);
                                s_adjs[j] = pj;
                                s_adjdeg[j] = (ldg_i(g.rp + pj + 1) & kMask) - (ldg_i(g.rp + pj) & kMask);
                            }
                        }
                        __syncthreads();
                    }
                    tick(2);
                    // Items of level l: the down segment, then the up frontier, then
                    // removal targets.  resolve() issues everything an item needs as
                    // one round of independent loads.
                    auto resolve = [&](int q, int &x, int &meta, double &c0, double &c1, double &c2,
                                       int2 &r, uint32_t &mk) -> bool {
                        if (q < nDl) {
                            const int idx = b0 + q;
                            x = Dv[idx];
                            const double2 s2 = st.sd[x];
                            c0 = s2.x;                // sigma (new)
                            c1 = s2.y;                // delta (old)
                            c2 = Dsig[idx];
                            const int od = Dold[idx];
                            meta = (((od & kOldMask) == l) ? kMetaNotPulled : 0) | ((od < 0) ? kMetaExt : 0) |
                                   ((ldg_i(g.rp + x) < 0) ? kMetaNew : 0);
                            r = row_of(g, x, lim);
                            st_bytes += 8 + 8;  // row bounds, delta read
                            return true;
                        }
                        const int qi = q - nDl;
                        x = -1;
                        if (qi < ucnt)
                            x = (qi < kUcap) ? s_un[ucur_sel][qi] : Ucur[qi - kUcap];
                        else if (Rl[qi - ucnt] == l)
                            x = Rv[qi - ucnt];
                        if (x < 0) return false;
                        // the dedup claim and the loads are issued together
                        const uint32_t prev = atomicMax(mark + x, E | kUpDone);
                        const double gxs = __ldcg(dacc + x);  // Ddelta / sigma (complete; helpers add via L2)
                        const double2 s2 = st.sd[x];
                        const double sx = s2.x, odl = s2.y;
                        const double gx = __dmul_rn(sx, gxs);
                        const bool usemask = l == 2 && mok;  // level-1 predecessors from the mask
                        const int2 rr = (push && !usemask) ? row_of(g, x, lim) : make_int2(0, 0);
                        mk = usemask ? mask[x] : 0u;
                        if (prev != mU) return false;  // a duplicate: the first claimant processes
                        meta = kMetaUp | (usemask ? kMetaMask : 0);
                        c0 = sx;
                        c1 = gx;
                        c2 = odl;
                        st_bytes += 8 + (usemask ? 4 : 0);  // Ddelta read
                        r = (push && gx != 0.0) ? rr : make_int2(0, 0);
                        if (gx == 0.0) mk = 0u;
                        return true;
                    };
                    auto inlane = [&](int x, int meta, double c0, double c1, double c2, int2 r, uint32_t mk) {
                        const bool wantpush = push && r.y > r.x;
                        if (meta & kMetaMask) {  // level 2: predecessors = set bits (root's row order)
                            for (uint32_t b = mk; b; b &= b - 1) {
                                const int pp = s_adjs[__ffs(b) - 1];
                                up_visit(c1, c0, pp, 0.0, mark[pp]);
                            }
                            up_finish(x, c1, c2);
                        } else if (meta & kMetaUp) {
                            if (wantpush) {
                                const double wx = __ddiv_rn(c1, c0);  // Ddelta[x] / sigma[x]
                                for (int j = r.x; j < r.y; j += kRowUnroll) {
                                    int y[kRowUnroll], dy[kRowUnroll];
                                    uint32_t mp[kRowUnroll], oc[kRowUnroll];
#pragma unroll
                                    for (int u = 0; u < kRowUnroll; ++u)
                                        y[u] = (j + u < r.y) ? ldg_i(g.col + j + u) : -1;
#pragma unroll
                                    for (int u = 0; u < kRowUnroll; ++u) dy[u] = (y[u] >= 0) ? st.d[y[u]] : kInf;
#pragma unroll
                                    for (int u = 0; u < kRowUnroll; ++u) {
                                        const bool pr = y[u] >= 0 && dy[u] == l - 1;
                                        mp[u] = pr ? mark[y[u]] : 0xffffffffu;
                                    }
#pragma unroll
                                    for (int u = 0; u < kRowUnroll; ++u)
                                        if (y[u] >= 0 && dy[u] == l - 1) {
                                            atomicAdd(dacc + y[u], wx);
                                            st_bytes += 24;
                                        }
#pragma unroll
                                    for (int u = 0; u < kRowUnroll; ++u)
                                        oc[u] = (mp[u] < E) ? atomicMax(mark + y[u], mU) : 0xffffffffu;
#pragma unroll
                                    for (int u = 0; u < kRowUnroll; ++u)
                                        if (oc[u] < E) {
                                            const int pos = atomicAdd(&s_ucnt2[ucur_sel ^ 1], 1);
                                            if (pos < kUcap)
                                                s_un[ucur_sel ^ 1][pos] = y[u];
                                            else
                                                Unext[pos - kUcap] = y[u];
                                        }
                                }
                                (l == 2 ? sc_up2 : sc_up3) += r.y - r.x;
                                st_bytes += 8 + 8ull * (r.y - r.x);
                            }
                            up_finish(x, c1, c2);
                        } else {
                            double dn = 0.0;
                            row_walk(g, st, nullptr, r, [&](int dy) { return dy == l + 1; },
                                     [&](int, int dy, double2 q, uint32_t) { dn += dpull_visit(c0, dy, q.x, q.y); });
                            sc_dpull += r.y - r.x;
                            st_bytes += 8ull * (r.y - r.x);
                            if (wantpush && (meta & kMetaExt)) {  // some predecessor outside D
                                row_walk(g, st, mark, r, [&](int dp) { return dp == l - 1; },
                                         [&](int pp, int dp, double2 q, uint32_t mp) {
                                             if (dp == l - 1)
                                                 dpush_visit(x, c0, dn, c1, c2, meta, pp, q.x, mp);
                                         });
                                sc_dpush += r.y - r.x;
                                (void)0;  // second walk of the same row: one pass in the byte model
                            }
                            d_finish(x, dn, c1);
                        }
                    };
                    // long row t of the chunk in I (level-2 rows resolved against adj(root)
                    // carry no entries of their own)
                    auto put_row = [&](int t, int x, int meta, double c0, double c1, double c2, int beg, int len,
                                       uint32_t mk) {
                        int elen = len;
                        if (meta & kMetaMask) {  // level 2 via the mask
                            if (mk) s_l1[atomicAdd(&s_nl1, 1)] = t;
                            elen = 0;
                        } else if ((meta & kMetaUp) && l == 2 && s_ds >= 0 && s_ds * (33 - __clz(len)) < len) {
                            // level 2 without masks: resolve against adj(root) by search
                            s_l1[atomicAdd(&s_nl1, 1)] = t;
                            elen = 0;
                        }
                        if (!(meta & (kMetaUp | kMetaExt))) s_noext = 1;  // a down row without pushes
                        I.mk[t] = mk;
                        I.v[t] = x;
                        I.meta[t] = meta;
                        I.beg[t] = beg;
                        I.off[t + 1] = elen;
                        I.acc[t] = 0.0;
                        I.c0[t] = c0;
                        I.c1[t] = c1;
                        I.c2[t] = c2;
                    };
                    XRow *Xw = a.ws.X + (size_t)wk * kXcap;
                    auto split_range = [&](int q0, int q1, bool small_inlane, bool defer) {
                        for (int q = q0 + tid; q < q1; q += kBlock) {
                            int x, meta = 0;
                            double c0 = 0.0, c1 = 0.0, c2 = 0.0;
                            int2 r = make_int2(0, 0);
                            uint32_t mk = 0u;
                            if (!resolve(q, x, meta, c0, c1, c2, r, mk)) continue;
                            const int len = r.y - r.x;
                            if (small_inlane && len <= kSmallDeg) {
                                inlane(x, meta, c0, c1, c2, r, mk);
                                continue;
                            }
                            const int t = atomicAdd(&s_nbigI, 1);
                            if (t >= kChunk) {  // shared list full: a later chunk, or in-lane
                                const bool up = (meta & kMetaUp) != 0;
                                const int xi = defer ? atomicAdd(&s_nx[up ? 1 : 0], 1) : kXcap;
                                if (xi < kXcap / 2) {  // down rows from the front, up rows from the back
                                    XRow &w = Xw[up ? kXcap - 1 - xi : xi];
                                    w.x = x;
                                    w.meta = meta;
                                    w.beg = r.x;
                                    w.len = len;
                                    w.c0 = c0;
                                    w.c1 = c1;
                                    w.c2 = c2;
                                    w.mk = mk;
                                } else {
                                    inlane(x, meta, c0, c1, c2, r, mk);
                                }
                                continue;
                            }
                            put_row(t, x, meta, c0, c1, c2, r.x, len, mk);
                        }
                    };
                    // small levels (<= one item per thread): short rows in-lane;
                    // large levels: every row through the flattened pass, in chunks
                    const int total = nDl + ucnt + rcnt;
                    const bool small_level = total <= kBlock || a.lowdeg;
                    // wide levels of up to wide_inlane items per thread: short rows in-lane
                    // in one pass, long rows through chunks of kChunk (the first in I, the
                    // rest deferred in Xw); wider levels: every row chunked
                    const bool wide = !small_level && total <= a.wide_inlane * kBlock;
                    const int step = (small_level || wide) ? total : kChunk;
                    bool first_barrier = true;
                    for (int cb = 0; cb < total; cb += step) {
                        const int ce = min(total, cb + step);
                        int nDb = 0;
                        const int nblk5 = (total + a.hd_block - 1) / a.hd_block;
                        if (wide && a.help.word && nblk5 >= a.he_min && worth(nblk5)) {
                            // the in-lane pass as help blocks (kind 5): every long row is
                            // deferred to Xw (the owner's chunks below), appends via gU
                            const int nl = min(ucnt, kUcap);
                            for (int i = tid; i < nl; i += kBlock) Bq[i] = s_un[ucur_sel][i];
                            UpCtx uc;
                            uc.g = g;
                            uc.st = st;
                            uc.mark = mark;
                            uc.dacc = dacc;
                            uc.bc = a.bc;
                            uc.mask = mask;
                            uc.Dv = Dv;
                            uc.Dold = Dold;
                            uc.Rv = Rv;
                            uc.Rl = Rl;
                            uc.Ul = Bq;
                            uc.Uo = Ucur;
                            uc.Dsig = Dsig;
                            uc.adjs = s_adjs;
                            uc.gU = a.help.gU + (size_t)wk * n;
                            uc.gapp = a.help.gapp + wk;
                            uc.xcnt = a.help.gbig + 2 * wk;
                            uc.X = Xw;
                            uc.l = l;
                            uc.b0 = b0;
                            uc.nDl = nDl;
                            uc.ucnt = ucnt;
                            uc.g0 = g0;
                            uc.lim = lim;
                            uc.mok = mok;
                            uc.E = E;
                            uc.mU = mU;
                            uc.mD = mD;
                            if (tid == 0) {
                                HelpCtx cx;
                                cx.root_slot = slot;
                                cx.l = l;
                                cx.g0 = g0;
                                cx.lim = lim;
                                cx.cnt = total;
                                cx.nblocks = nblk5;
                                cx.E2 = nDl;
                                cx.E = E;
                                cx.kind = 5;
                                cx.lb = b0;
                                cx.mvalid = mok;
                                cx.aux = ucnt | ((Ucur == Ub) ? (1 << 30) : 0);
                                a.help.ctx[wk] = cx;
                                a.help.done[wk] = 0;
                                a.help.gapp[wk] = 0;
                                a.help.gbig[2 * wk] = 0;
                                a.help.gbig[2 * wk + 1] = 0;
                            }
                            __syncthreads();  // the frontier copy is written; one release fence publishes it
                            if (tid == 0) {
                                __threadfence();
                                atomicAdd(stat_lane(a.stats) + kStHelpReq, 1ull);
                                atomicAdd(stat_lane(a.stats) + kStHelpBlkAll, (unsigned long long)nblk5);
                                atomicAdd(stat_lane(a.stats) + kStUpPass, 1ull);
                                hseq = (hseq + 1) & 0xFFFF;
                                atomicExch(a.help.word + wk, help_pack(1, nblk5, 0, hseq));
                                if (nblk5 >= a.busy_min) atomicAdd(a.help.roots_left + 1, 1);
                            }
                            for (;;) {  // the owner takes blocks too
                                if (tid == 0) {
                                    const unsigned long long w = atomicAdd(a.help.word + wk, 1ull << 16);
                                    s_hb = help_next(w) < nblk5 ? help_next(w) : -1;
                                }
                                __syncthreads();
                                const int b = s_hb;
                                __syncthreads();
                                if (b < 0) break;
                                ++own_blk;
                                up_block(uc, b * a.hd_block, min(total, (b + 1) * a.hd_block), st_bytes,
                                         sc_up3);  // ends with a barrier
                                if (tid == 0) {
                                    __threadfence();
                                    atomicAdd(a.help.done + wk, 1);
                                }
                            }
                            trace(6, 5, own_blk | (nblk5 << 16));
                            own_blk = 0;
                            if (tid == 0) {  // wait for the helpers' blocks, then close
                                while (atomicAdd(a.help.done + wk, 0) < nblk5) __nanosleep(256);
                                atomicExch(a.help.word + wk, help_pack(0, 0, 0, hseq));
                                if (nblk5 >= a.busy_min) atomicSub(a.help.roots_left + 1, 1);
                                __threadfence();
                                s_nx[0] = __ldcg(a.help.gbig + 2 * wk);
                                s_nx[1] = __ldcg(a.help.gbig + 2 * wk + 1);
                                s_nbigI = 0;
                            }
                            __syncthreads();
                            const int gc = __ldcg(a.help.gapp + wk);  // merge the global appends
                            for (int i = tid; i < gc; i += kBlock) {
                                const int y = __ldcg(uc.gU + i);
                                const int pos = atomicAdd(&s_ucnt2[ucur_sel ^ 1], 1);
                                if (pos < kUcap)
                                    s_un[ucur_sel ^ 1][pos] = y;
                                else
                                    Unext[pos - kUcap] = y;
                            }
                            __syncthreads();
                        } else {
                            if (cb < nDl) {  // down rows first: their pull precedes their push
                                split_range(cb, min(ce, nDl), small_level || wide, wide);
                                __syncthreads();
                                nDb = min(s_nbigI, kChunk);
                            }
                            split_range(max(cb, nDl), ce, small_level || wide, wide);
                            __syncthreads();
                        }
                        if (first_barrier) {  // the current list's count was read last level
                            first_barrier = false;
                            if (tid == 0) s_ucnt2[ucur_sel] = 0;
                        }
                        tick(6);
                        trace(10, 0, min(s_nbigI, kChunk));  // chunk split done: long rows
                        int nb = min(s_nbigI, kChunk);
                        int xdn = 0, xun = 0;  // deferred down / up rows already loaded
                        for (;;) {  // the chunk in I, then (wide levels) the deferred rows
                        if (nb > 0) {
                            chunk_scan(I.off, nb);  // off[0..nb], ends with a barrier
                            tick(7);
                            trace(11, 0, I.off[nDb]);  // C1 entries
                            auto colf = [&](int t, int e) { return ldg_i(g.col + I.beg[t] + e - I.off[t]); };
                            // --- C1: delta pull of the long down rows (Eq. (2)) ---
                            const int E1 = I.off[nDb];
                            auto c1_pass = [&](int e0, int e1) {
                                flat_entries(I.off, nb, e1, colf, st, nullptr, [&](int dy) { return dy == l + 1; },
                                             I.acc, [&](int t, int, int dy, double2 q, uint32_t) {
                                                 sc_dpull++;
                                                 st_bytes += 8;
                                                 return dpull_visit(I.c0[t], dy, q.x, q.y);
                                             }, e0);
                            };
                            const int nblk1 = (E1 + a.he_entries - 1) / a.he_entries;
                            if (E1 > 0 && a.help.word && nblk1 >= a.he_min && worth(nblk1)) {
                                // publish the pull rows; helpers add per-row partial sums
                                // into the mirror's acc (delta: rounding order is free)
                                ChunkSmem *mir = a.help.mir + wk;
                                for (int t = tid; t < nDb; t += kBlock) {
                                    mir->v[t] = I.v[t];
                                    mir->meta[t] = I.meta[t];
                                    mir->beg[t] = I.beg[t];
                                    mir->off[t + 1] = I.off[t + 1];
                                    mir->acc[t] = 0.0;
                                    mir->c0[t] = I.c0[t];
                                }
                                if (tid == 0) {
                                    HelpCtx cx;
                                    cx.root_slot = slot;
                                    cx.l = l;
                                    cx.g0 = g0;
                                    cx.lim = lim;
                                    cx.cnt = nDb;
                                    cx.nblocks = nblk1;
                                    cx.E2 = E1;
                                    cx.E = E;
                                    cx.kind = 2;
                                    cx.lb = 0;
                                    cx.mvalid = 0;
                                    mir->off[0] = 0;
                                    a.help.ctx[wk] = cx;
                                    a.help.done[wk] = 0;
                                }
                                __syncthreads();
                                if (tid == 0) {
                                    __threadfence();
                                    atomicAdd(stat_lane(a.stats) + kStHelpReq, 1ull);
                                    atomicAdd(stat_lane(a.stats) + kStHelpBlkAll, (unsigned long long)nblk1);
                                    hseq = (hseq + 1) & 0xFFFF;
                                    atomicExch(a.help.word + wk, help_pack(1, nblk1, 0, hseq));
                                    if (nblk1 >= a.busy_min) atomicAdd(a.help.roots_left + 1, 1);  // open wide requests
                                }
                                for (;;) {  // the owner takes blocks too
                                    if (tid == 0) {
                                        const unsigned long long w = atomicAdd(a.help.word + wk, 1ull << 16);
                                        s_hb = help_next(w) < nblk1 ? help_next(w) : -1;
                                    }
                                    __syncthreads();
                                    const int b = s_hb;
                                    __syncthreads();
                                    if (b < 0) break;
                                    ++own_blk;
                                    c1_pass(b * a.he_entries, min(E1, (b + 1) * a.he_entries));  // ends with a barrier
                                    if (tid == 0) atomicAdd(a.help.done + wk, 1);
                                }
                                trace(6, 2, own_blk | (nblk1 << 16));
                                own_blk = 0;
                                if (tid == 0) {  // wait for the helpers' blocks, then close
                                    while (atomicAdd(a.help.done + wk, 0) < nblk1) __nanosleep(256);
                                    atomicExch(a.help.word + wk, help_pack(0, 0, 0, hseq));
                                    if (nblk1 >= a.busy_min) atomicSub(a.help.roots_left + 1, 1);
                                    __threadfence();
                                }
                                __syncthreads();
                                for (int t = tid; t < nDb; t += kBlock) I.acc[t] += __ldcg(&mir->acc[t]);
                                __syncthreads();
                            } else if (E1 > 0) {
                                c1_pass(0, E1);
                            }
                            tick(8);
                            trace(12, 0, I.off[nb]);  // C2 (before compaction)
                            // --- C2: pushes towards level l-1 (down rows only if they have a
                            // predecessor outside D: drop the others from the offsets) ---
                            if (push && s_noext) {
                                constexpr int per = (kChunk + kBlock - 1) / kBlock;
                                int ln[per];
#pragma unroll
                                for (int k = 0; k < per; ++k) {
                                    const int t = tid + k * kBlock;
                                    ln[k] = (t < nb && (I.meta[t] & (kMetaUp | kMetaExt))) ? I.off[t + 1] - I.off[t] : 0;
                                }
                                __syncthreads();
#pragma unroll
                                for (int k = 0; k < per; ++k) {
                                    const int t = tid + k * kBlock;
                                    if (t < nb) I.off[t + 1] = ln[k];
                                }
                                __syncthreads();
                                chunk_scan(I.off, nb);
                            }
                            const int E2 = I.off[nb];
                            const int nblk = (E2 + a.he_entries - 1) / a.he_entries;
                            if (push && E2 > 0 && a.help.word && nblk >= a.he_min && worth(nblk)) {
                                // publish the chunk; idle workers help block by block
                                ChunkSmem *mir = a.help.mir + wk;
                                for (int t = tid; t < nb; t += kBlock) {
                                    mir->v[t] = I.v[t];
                                    mir->meta[t] = I.meta[t];
                                    mir->beg[t] = I.beg[t];
                                    mir->off[t + 1] = I.off[t + 1];
                                    mir->acc[t] = I.acc[t];
                                    mir->c0[t] = I.c0[t];
                                    mir->c1[t] = I.c1[t];
                                    mir->c2[t] = I.c2[t];
                                }
                                HelpCtx cx;
                                cx.root_slot = slot;
                                cx.l = l;
                                cx.g0 = g0;
                                cx.lim = lim;
                                cx.cnt = nb;
                                cx.nblocks = nblk;
                                cx.E2 = E2;
                                cx.E = E;
                                cx.kind = 0;
                                cx.lb = 0;
                                cx.mvalid = 0;
                                if (tid == 0) {
                                    mir->off[0] = 0;
                                    a.help.ctx[wk] = cx;
                                    a.help.done[wk] = 0;
                                    a.help.gapp[wk] = 0;
                                }
                                __syncthreads();  // the chunk is written; one release fence publishes it
                                if (tid == 0) {
                                    __threadfence();
                                    atomicAdd(stat_lane(a.stats) + kStHelpReq, 1ull);
                                    atomicAdd(stat_lane(a.stats) + kStHelpBlkAll, (unsigned long long)nblk);
                                    hseq = (hseq + 1) & 0xFFFF;
                                    atomicExch(a.help.word + wk, help_pack(1, nblk, 0, hseq));
                                    if (nblk >= a.busy_min) atomicAdd(a.help.roots_left + 1, 1);  // open wide requests
                                }
                                int32_t *gU = a.help.gU + (size_t)wk * n;
                                int *gapp = a.help.gapp + wk;
                                for (;;) {  // the owner takes blocks too
                                    if (tid == 0) {
                                        const unsigned long long w = atomicAdd(a.help.word + wk, 1ull << 16);
                                        s_hb = help_next(w) < nblk ? help_next(w) : -1;
                                    }
                                    __syncthreads();
                                    const int b = s_hb;
                                    __syncthreads();
                                    if (b < 0) break;
                                    ++own_blk;
                                    help_run_block<false>(I, b * a.he_entries, min(E2, (b + 1) * a.he_entries), g,
                                                          st, mark, dacc, gU, gapp, cx, st_bytes);
                                    __syncthreads();  // (help_run_block ends with one too)
                                    if (tid == 0) {   // release by one thread after the CTA barrier
                                        __threadfence();
                                        atomicAdd(a.help.done + wk, 1);
                                    }
                                }
                                trace(6, 0, own_blk | (nblk << 16));
                                own_blk = 0;
                                if (tid == 0) {  // wait for the helpers' blocks, then close
                                    while (atomicAdd(a.help.done + wk, 0) < nblk) __nanosleep(256);
                                    atomicExch(a.help.word + wk, help_pack(0, 0, 0, hseq));
                                    if (nblk >= a.busy_min) atomicSub(a.help.roots_left + 1, 1);
                                    __threadfence();
                                }
                                __syncthreads();
                                const int gc = __ldcg(gapp);  // merge the global appends
                                for (int i = tid; i < gc; i += kBlock) {
                                    const int y = __ldcg(gU + i);
                                    const int pos = atomicAdd(&s_ucnt2[ucur_sel ^ 1], 1);
                                    if (pos < kUcap)
                                        s_un[ucur_sel ^ 1][pos] = y;
                                    else
                                        Unext[pos - kUcap] = y;
                                }
                                __syncthreads();
                            } else if (push && E2 > 0)
                                flat_push<false>(  // pushes need no sigma of the target; claims batched
                                    I.off, nb, E2, colf, st, mark, E, [&](int dp) { return dp == l - 1; },
                                    [&](int t, int pp, int dp, uint32_t mp) -> uint32_t {
                                        (l == 2 ? sc_up2 : sc_up3)++;
                                        const int meta = I.meta[t];
                                        if (meta & kMetaUp) st_bytes += 8;  // D rows: counted by their C1 pull
                                        if (dp != l - 1) return 0u;
                                        if (meta & kMetaUp) {
                                            atomicAdd(dacc + pp, __ddiv_rn(I.c1[t], I.c0[t]));
                                            st_bytes += 24;
                                            return mp >= E ? 0u : mU;
                                        }
                                        if (mp == mD) return 0u;
                                        double dlt = __ddiv_rn(1.0 + I.acc[t], I.c0[t]);
                                        if ((meta & kMetaNotPulled) &&
                                            !((meta & kMetaNew) && new_edge(g, I.v[t], pp, g0, lim)))
                                            dlt = __dsub_rn(dlt, __ddiv_rn(1.0 + I.c1[t], I.c2[t]));
                                        atomicAdd(dacc + pp, dlt);
                                        st_bytes += 24;
                                        return mp >= E ? 0u : mU;
                                    },
                                    [&](int y) {  // claimed: the next up frontier
                                        const int pos = atomicAdd(&s_ucnt2[ucur_sel ^ 1], 1);
                                        if (pos < kUcap)
                                            s_un[ucur_sel ^ 1][pos] = y;
                                        else
                                            Unext[pos - kUcap] = y;
                                    });
                            tick(9);
                            trace(13, 0, s_nl1);
                            // --- C3: level-2 rows resolved against adj(root) ---
                            const int nl1 = s_nl1;
                            if (nl1 > 0) {
                                const int ds = s_ds, npairs = nl1 * ds;
                                for (int j = tid; j < ds; j += kBlock) s_l1acc[j] = 0.0;
                                __syncthreads();
                                // Ddelta[p] += sigma[p] * sum_x Ddelta[x] / sigma[x] over the
                                // level-2 rows x adjacent to level-1 vertex p (per-p sums in
                                // shared memory, one global update per p)
                                for (int qq = tid; qq < npairs; qq += kBlock) {
                                    const int li = qq / ds, j = qq - li * ds;
                                    const int t = s_l1[li];
                                    const int x = I.v[t], pp = s_adjs[j];
                                    bool adj;
                                    if (I.meta[t] & kMetaMask) {
                                        adj = (I.mk[t] >> j) & 1u;
                                    } else {
                                        const int degx = (ldg_i(g.rp + x + 1) & kMask) - (ldg_i(g.rp + x) & kMask);
                                        adj = (s_adjdeg[j] < degx) ? adjacent_visible(g, pp, x, lim)
                                                                   : adjacent_visible(g, x, pp, lim);
                                        st_bytes += 32;
                                    }
                                    if (adj) atomicAdd(&s_l1acc[j], __ddiv_rn(I.c1[t], I.c0[t]));
                                }
                                __syncthreads();
                                for (int j = tid; j < ds; j += kBlock) {
                                    const double w = s_l1acc[j];
                                    if (w != 0.0) {
                                        const int pp = s_adjs[j];
                                        atomicAdd(dacc + pp, w);
                                        st_bytes += 24;
                                        claim_up(pp, mark[pp]);
                                    }
                                }
                                __syncthreads();
                            }
                            tick(4);
                            trace(14, 0, nb);
                            // --- epilogue of the long rows (Alg. 8 fused) ---
                            for (int t = tid; t < nb; t += kBlock) {
                                if (I.meta[t] & kMetaUp)
                                    up_finish(I.v[t], I.c1[t], I.c2[t]);
                                else
                                    d_finish(I.v[t], I.acc[t], I.c1[t]);
                            }
                            __syncthreads();
                        }
                        if (tid == 0) {
                            s_nbigI = 0;
                            s_nl1 = 0;
                            s_noext = 0;
                            s_hopen = hopen_pf;
                        }
                        __syncthreads();
                        if (!wide) break;
                        const int nxd = min(s_nx[0], kXcap / 2), nxu = min(s_nx[1], kXcap / 2);
                        const bool dn = xdn < nxd;  // deferred down rows first (own chunks: C1 then C2)
                        if (!dn && xun >= nxu) break;
                        const int m = dn ? min(kChunk, nxd - xdn) : min(kChunk, nxu - xun);
                        for (int t = tid; t < m; t += kBlock) {
                            const XRow &w = Xw[dn ? xdn + t : kXcap - 1 - (xun + t)];
                            put_row(t, w.x, w.meta, w.c0, w.c1, w.c2, w.beg, w.len, w.mk);
                        }
                        if (dn) xdn += m; else xun += m;
                        if (tid == 0) atomicAdd(stat_lane(a.stats) + kStDeferred, (unsigned long long)m);
                        nb = m;
                        nDb = dn ? m : 0;
                        __syncthreads();
                        }  // deferred chunks
                        if (wide && tid == 0) {
                            s_nx[0] = 0;
                            s_nx[1] = 0;
                        }
                        __syncthreads();
                    }  // chunks
                    tick(3);
                    // the chunk loop ended with a barrier: every append of this level is in
                    ucnt = s_ucnt2[ucur_sel ^ 1];
                    if (tid == 0) s_st[0] += ucnt;
                    int *t = Ucur;
                    Ucur = Unext;
                    Unext = t;
                    ucur_sel ^= 1;
                    tick(5);
                }
                // any up vertices left at level 0 would be the root: never produced
                if (a.scen && tid == 0)  // Fig. 2 / Fig. 4 record: case | touched << 2 | |D| << 33
                    a.scen[(size_t)ins * a.k_loc + slot] = (long long)(((unsigned long long)dtotal << 33) |
                                                                       ((s_st[0] - s_touch0) << 2) |
                                                                       (s_wcnt[1] ? 3u : 2u));
            }
            trace(4, 0, 0);
            ins = wend;
            __syncthreads();  // the counters are reset by the next window
        }
        if (a.help.word && tid == 0) atomicSub(a.help.roots_left, 1);
        if (a.root_prof && tid == 0) {
            unsigned long long t1;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
            unsigned long long *rp4 = a.root_prof + 6 * (size_t)slot;
            rp4[0] = s_prof[0];
            rp4[1] = t1;
            rp4[2] = s_prof[1];
            rp4[3] = s_st[0] - s_prof[2];
            rp4[4] = (unsigned long long)sc_down + sc_rem + sc_dpull + sc_dpush + sc_up2 + sc_up3 - s_prof[3];
            rp4[5] = s_st[5] + s_st[6] - s_prof[4];
        }
    }
    // ---- out of roots: help the passes of workers still running ----
    if (a.help.word) {
        int cur_owner = -1, cur_seq = -1;
        if (tid == 0) atomicAdd(a.help.roots_left + 2, 1);  // one more idle worker
        for (;;) {
            const int r = help_step(true, cur_owner, cur_seq);
            if (r == -2) break;
            if (r < 0) __nanosleep(1000);
        }
    }
    if (tid == 0) {
        a.ws.wepoch[wk] = epoch;
        if (s_st[2]) atomicAdd(stat_lane(a.stats) + kStCase1, s_st[2]);
        if (s_st[3]) atomicAdd(stat_lane(a.stats) + kStCase2, s_st[3]);
        if (s_st[4]) atomicAdd(stat_lane(a.stats) + kStCase3, s_st[4]);
        if (s_st[0]) atomicAdd(stat_lane(a.stats) + kStTouched, s_st[0]);
        if (s_st[1]) atomicAdd(stat_lane(a.stats) + kStDown, s_st[1]);
        if (s_st[5]) atomicAdd(stat_lane(a.stats) + kStLevDown, s_st[5]);
        if (s_st[6]) atomicAdd(stat_lane(a.stats) + kStLevUp, s_st[6]);
        for (int q = 0; q < 10; ++q)
            if (tm_ph[q]) atomicAdd(stat_lane(a.stats) + kStTime0 + q, tm_ph[q]);
    }
    const unsigned long long sc[6] = {sc_down, sc_rem, sc_dpull, sc_dpush, sc_up2, sc_up3};
    unsigned long long tot = 0;
#pragma unroll
    for (int q = 0; q < 6; ++q) {
        tot += sc[q];
        stat_add_warp(a.stats, kStPhase0 + q, sc[q]);
    }
    stat_add_warp(a.stats, kStScanned, tot);
    stat_add_warp(a.stats, kStBytes, st_bytes);
}

}  // namespace

#define DBC_CAT2(a, b) a##b
#define DBC_CAT(a, b) DBC_CAT2(a, b)
#ifndef DBC_LAUNCH_SUFFIX
#define DBC_LAUNCH_SUFFIX DBC_BLOCK
#endif
void DBC_CAT(launch_update_, DBC_LAUNCH_SUFFIX)(const UpdateArgs &a, int workers, cudaStream_t s) {
    update_kernel<<<workers, kBlock, 0, s>>>(a);
}

}  // namespace dbc
