// update_lean.cu -- K2/K3/K4 for ONE (root, insertion) at a time: the
// per-insertion update of the paper's structure (Sec. III, P:244-252;
// Sec. IV "reinserted into the graph one at a time").  Used for Mode S
// (one launch per insertion), DBC_FLAG_NO_MERGE batches, single-edge calls and
// the scenario log; window-merged batches (R18) run update.cu.
//
// Per job (root s, insertion i = (u, v), the graph as of insertion i):
//  classify (K2): Case 1 iff d(u) == d(v) (both unreachable
//      included): nothing changes.  Else u_high = the closer endpoint, u_low the
//      other; Case 3 iff d(u_low) > d(u_high) + 1 (u_low unreachable included).
//  seed (A2; replaces Alg. 3's O(n) init): Case 3 lowers u_low to
//      d(u_high) + 1 remembering its old distance; D = {u_low}.
//  down (K3; Alg. 2 stage 2): level-synchronous from u_low's level L.
//      Every w of level L gets sigma[w] = sum of sigma[x] over x in adj(w) with
//      d[x] = L - 1 -- a pull in canonical adjacency order (R5; a
//      parallel reduction is kept only when the sum is below 2^53, where every
//      order is exact, else the row is re-summed in order) -- and every
//      neighbour y with d[y] > L + 1 is pulled up to L + 1 (atomicMin; the
//      first lowerer records the old d), every neighbour with d[y] = L + 1 is
//      claimed (epoch-tagged flag: Alg. 2's t[y] = down) for level L + 1.
//  removal (A4 step 0, Case 3 only): each pulled-up w of finite old level gives
//      every old predecessor x not in D (d[x] = old d(w) - 1) the old
//      contribution back: Ddelta[x] -= sigma[x] / sigma_old(w) * (1 + delta_old(w)).
//  up (K4; Alg. 2 stage 3; Alg. 8 fused): for l from the
//      deepest touched level down to 1,
//        D vertex x: delta_new = sum over successors y (d[y] = l + 1) of
//          sigma[x] / sigma[y] * (1 + delta[y]) (Eq. (2), by pull);
//          BC[x] += delta_new - delta_old; each predecessor p not in D gets
//          Ddelta[p] += sigma[p] * ((1 + delta_new) / sigma_new
//                                  - (1 + delta_old) / sigma_old)
//          -- the old term only over an edge that existed before (never over
//          the new edge: Alg. 2's guard "v != u_high or w != u_low", P:216,
//          DESIGN.md R7) and not for a pulled-up x (its old predecessors were
//          handled by the removal pass);
//        up vertex x (t[x] = up): delta[x] += Ddelta[x], BC[x] += Ddelta[x], and
//          for l >= 2 every predecessor p gets Ddelta[p] += sigma[p] / sigma[x] *
//          Ddelta[x].  At l = 1 the only predecessor is s, whose delta is never
//          used.
//      The accumulator holds Ddelta[p] / sigma[p] (sigma[p] does not change for
//      p outside D), so a push needs no gather of the target's sigma and an up
//      vertex forwards its own accumulator value unchanged.
//
// B200 mapping: a persistent grid of worker CTAs (kBlock threads, all resident)
// takes roots from a counter; a worker walks the launch's insertions for its
// root in order.  A level is processed in chunks of up to kLCap items whose
// rows are flattened over the CTA (every thread takes kLU consecutive entries;
// gathers are issued together: col, then d, then sigma / (sigma, delta) / the
// claim flag only where the d test passes).  A wide pass (a hub-heavy level of
// one root: thousands of rows, 10^5 entries) is published on a help board and
// the workers that have run out of roots take blocks of kHelpBlk entries --
// one root's level then runs on many SMs.  All mutable state is read through
// L2 (ld.cg): helpers on other SMs write it with atomics.  Per job nothing is
// O(n): scratch is epoch-tagged and the accumulator is reset by the vertex that
// consumes it.
#include "dbc_internal.cuh"

namespace dbc {

namespace {

constexpr int kLCap = 512;        // items per chunk
constexpr int kLStash = 512;      // D-row predecessor pushes staged per chunk
constexpr int kLWin = kBlock < 256 ? kBlock : 256;  // insertions classified at once
constexpr int kLAdj = 256;        // longest root row cached (level-2 shortcut)
#ifndef DBC_LEAN_LU
#define DBC_LEAN_LU 4
#endif
#ifndef DBC_LEAN_HELPBLK
#define DBC_LEAN_HELPBLK 2048
#endif
#ifndef DBC_LEAN_HELPMIN
#define DBC_LEAN_HELPMIN 3
#endif
constexpr int kLU = DBC_LEAN_LU;  // consecutive entries per thread per step
constexpr uint32_t kLD = 3u;      // mark: in D (t = down).  kLD > kLUp: an up claim
constexpr uint32_t kLUp = 1u;     // mark: up (t = up)        never overrides a D mark
constexpr int kHelpBlk = DBC_LEAN_HELPBLK;  // entries per help block
constexpr int kHelpMinBlk = DBC_LEAN_HELPMIN;  // passes of at least this many blocks are published
constexpr int kLEnt = 1536;       // entries whose contributions are kept for an in-order row sum
constexpr int kSpecEntries = 2 * kBlock * kLU;  // passes up to this size gather speculatively
// Shared-memory copy of the job's D list (ids, old d, old sigma) for its first
// kDMir entries: the up phase's D rows and the removal pass read them without a
// global round trip.  Dynamic shared memory (kLDyn bytes).
constexpr int kDMir = kBlock * 2 < 1024 ? kBlock * 2 : 1024;
constexpr int kLDyn = kDMir * (int)(2 * sizeof(int) + sizeof(double));

// pass kinds (entry visitors)
enum : int { kPDown = 1, kPUp = 2, kPRem = 3, kPDRow = 4, kPDPush = 5 };

struct LeanSmem {
    int v[kLCap];
    int beg[kLCap];
    int off[kLCap + 1];
    int aux[kLCap];      // D index (D rows), target level (removal rows)
    double acc[kLCap];
    double c0[kLCap], c1[kLCap];
    int st_p[kLStash];
    short st_t[kLStash];
    int sc_t[kLCap];     // shortcut items of the chunk
    double ev[kLEnt];    // per-entry contribution of a local pass (rows summed in canonical order)
    int adjs[kLAdj];
    int wul[kLWin], wlev[kLWin], wq[kLWin];
    int nx[kLCap];       // the next down level's first kLCap vertices (mirror of Dv)
    int um[2][kLCap];    // the up lists' first kLCap vertices (mirrors of U0 / U1)
};

// A pass published for help (global memory, one per worker).
struct LeanBoard {
    unsigned long long word;  // bit 63 open | nblk << 40 | next << 16 | seq
    int done;                 // blocks finished
    int ctr;                  // append counter of the pass
    int low, rmin, rmax;      // down: a distance was lowered; removal: target level range
    int kind, slot, l, cnt, Etot, sel;  // sel: which up list receives appends
    uint32_t E, epoch;
    int ul, uh, pull;         // the job's insertion (D-row pushes skip the old term over it)
    int off[kLCap + 1];
    int beg[kLCap];
    int aux[kLCap];
    int v[kLCap];
    double c0[kLCap], c1[kLCap];
    double acc[kLCap];
};

__device__ __forceinline__ unsigned long long hb_pack(int open, int nblk, int next, int seq) {
    return ((unsigned long long)(open ? 1 : 0) << 63) | ((unsigned long long)(nblk & 0xFFFFF) << 40) |
           ((unsigned long long)(next & 0xFFFFF) << 16) | (unsigned long long)(seq & 0xFFFF);
}
__device__ __forceinline__ bool hb_open(unsigned long long w) { return (w >> 63) != 0; }
__device__ __forceinline__ int hb_nblk(unsigned long long w) { return (int)((w >> 40) & 0xFFFFF); }
__device__ __forceinline__ int hb_next(unsigned long long w) { return (int)((w >> 16) & 0xFFFFF); }
__device__ __forceinline__ int hb_seq(unsigned long long w) { return (int)(w & 0xFFFF); }

// Everything an entry visitor needs; counters / accumulators are generic
// pointers (shared memory for a local pass, the board for a published one).
struct PassCtx {
    int kind, l;                 // pass kind; the level L (down) or l (up)
    uint32_t E, mD, mU;          // epoch tag and marks of the job
    unsigned long long E64;      // epoch << 32 (lowering records)
    Root st;
    uint32_t *mark;
    unsigned long long *lowrec;
    double *dacc;
    int32_t *list, *list2;       // appends: Dv (down), an up list (up), Rv / Rl (removal)
    int *ctr;
    int *mir;                    // nullable: shared mirror of the list's entries [mbase, mbase + kLCap)
    int mbase;
    int mirbit;                  // its s_mirbad bit
    int *dmir;                   // nullable: shared copy of the D list (down passes of the owner)
    int *low, *rmin, *rmax;
    double *acc;                 // per-row sums (when ev == nullptr)
    double *ev;                  // per-entry contributions (a local pass of <= kLEnt entries)
    int ul, uh;                  // the job's insertion
    bool stash;                  // kPDRow: stage predecessors in shared memory (a local pass)
    unsigned long long *ptr;     // -DDBC_LEAN_PTRACE builds: step clocks of the traced root's up passes
    bool full;
    bool pull;                   // DBC_FLAG_PULL_DELTA: targets are only claimed (they pull)                   // scenario log: claim even over a zero push (Alg. 2's touched set)
};

__device__ __forceinline__ int block_excl_scan(int x, int *total) {
    __shared__ int ws[kWarps];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    int incl = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(kFull, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) ws[wid] = incl;
    __syncthreads();
    int base = 0, tot = 0;
#pragma unroll
    for (int w = 0; w < kWarps; ++w) {
        const int s = ws[w];
        base += (w < wid) ? s : 0;
        tot += s;
    }
    *total = tot;
    __syncthreads();
    return base + incl - x;
}

// Exclusive offsets of the chunk's row lengths (S.off[t+1] holds len t on
// entry); returns the total.  Ends with a barrier.
__device__ __forceinline__ int chunk_offsets(LeanSmem &S, int cnt) {
    if (cnt <= 32) {  // a narrow level: warp 0 scans alone (one barrier instead of three)
        __shared__ int s_tot;
        if (threadIdx.x < 32) {
            const int lane = threadIdx.x;
            const int x = lane < cnt ? S.off[lane + 1] : 0;
            int incl = x;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int y = __shfl_up_sync(kFull, incl, o);
                if (lane >= o) incl += y;
            }
            if (lane < cnt) S.off[lane + 1] = incl;
            if (lane == 31) s_tot = incl;
            if (lane == 0) S.off[0] = 0;
        }
        __syncthreads();
        return s_tot;
    }
    constexpr int per = kLCap / kBlock > 0 ? kLCap / kBlock : 1;
    int vals[per];
    int run = 0;
#pragma unroll
    for (int q = 0; q < per; ++q) {
        const int i = threadIdx.x * per + q;
        vals[q] = i < cnt ? S.off[i + 1] : 0;
        run += vals[q];
    }
    int tot;
    int ex = block_excl_scan(run, &tot);
#pragma unroll
    for (int q = 0; q < per; ++q) {
        const int i = threadIdx.x * per + q;
        ex += vals[q];
        if (i < cnt) S.off[i + 1] = ex;
    }
    if (threadIdx.x == 0) S.off[0] = 0;
    __syncthreads();
    return tot;
}

// what to gather for an entry with distance dy of row t: bit 0 (sigma, delta),
// bit 1 the claim flag
template <int K>
__device__ __forceinline__ int pass_sel(const PassCtx &c, const LeanSmem &S, int t, int dy) {
    switch (K) {
        case kPDown: return dy == c.l - 1 ? 1 : (dy == c.l + 1 ? 2 : 0);
        case kPUp: return dy == c.l - 1 ? 2 : 0;
        case kPRem: return dy == S.aux[t] ? 2 : 0;
        case kPDPush: return dy == c.l - 1 ? 2 : 0;
        default: return (dy == c.l + 1 ? 1 : 0) | ((c.l >= 2 && dy == c.l - 1) ? 2 : 0);  // kPDRow
    }
}

// everything a pass kind may gather (speculative gathers of a narrow pass)
template <int K>
__device__ __forceinline__ constexpr int pass_spec() {
    return K == kPDown ? 3 : (K == kPDRow ? 3 : 2);  // kPUp, kPRem, kPDPush: the flag
}

__device__ __forceinline__ void claim_append(const PassCtx &c, int y, uint32_t m) {
    if (atomicMax(c.mark + y, m) < c.E) {
        const int p = atomicAdd(c.ctr, 1);
        c.list[p] = y;
        if (c.mir && p - c.mbase < kLCap) c.mir[p - c.mbase] = y;
        if (c.dmir && p < kDMir) c.dmir[p] = y;
    }
}

// One entry (row t, neighbour y at distance dy; q / mk gathered per pass_sel),
// first half: the row's contribution (sigma for down rows, the delta term for
// D rows) and fire-and-forget updates; the atomics whose result matters are
// returned as requests -- *low: a lowering to l + 1 (Case 3), *claim: the mark
// to claim y with -- and issued by lean_pass for all of a thread's entries
// together (one round trip instead of one per entry).
template <int K>
__device__ __forceinline__ double pass_visit(const PassCtx &c, LeanSmem &S, int *s_nst, int t, int y, int dy,
                                             double2 q, uint32_t mk, uint32_t &bytes, bool *low,
                                             uint32_t *claim) {
    bytes += 8;
    switch (K) {
        case kPDown:
            if (dy == c.l - 1) {  // predecessor: sigma (pull, Alg. 2 line 14 / P:238)
                bytes += 8;
                return q.x;
            }
            if (dy > c.l + 1) {  // Case 3: pull y up to l + 1 (the first lowerer records the old d)
                *low = true;
                *claim = c.mD;
            } else if (dy == c.l + 1 && mk < c.E) {  // successor: t[y] = down
                *claim = c.mD;
            }
            return 0.0;
        case kPUp:  // up vertex: Ddelta[p] += sigma[p] / sigma[x] * Ddelta[x] (factored)
            if (dy == c.l - 1) {
                const double f = S.c0[t];
                if (f != 0.0) atomicAdd(c.dacc + y, f);
                bytes += 16;
                if (mk < c.E) *claim = c.mU;
            }
            return 0.0;
        case kPRem:  // an old predecessor outside D gets the old contribution back
            if (dy == S.aux[t] && mk != c.mD) {
                if (!c.pull) atomicAdd(c.dacc + y, S.c0[t]);
                bytes += 16;
                if (mk < c.E) *claim = c.mU;
            }
            return 0.0;
        case kPDPush:  // D row x: Ddelta[p] += sigma[p] * ((1 + delta_new) / sigma_new - old term)
            if (dy == c.l - 1 && mk != c.mD) {
                if (c.pull) {  // the predecessor pulls its own delta
                    if (mk < c.E) *claim = c.mU;
                    return 0.0;
                }
                const bool ne = S.v[t] == c.ul && y == c.uh;  // never an old term over the new edge
                const double w = ne ? S.c0[t] : __dsub_rn(S.c0[t], S.c1[t]);
                if (w != 0.0) atomicAdd(c.dacc + y, w);
                bytes += 16;
                if ((w != 0.0 || c.full) && mk < c.E) *claim = c.mU;
            }
            return 0.0;
        default:  // kPDRow: delta by pull; predecessors outside D staged for pushes
            if (dy == c.l + 1) {
                bytes += 16;
                return __dmul_rn(__ddiv_rn(S.c0[t], q.x), __dadd_rn(1.0, q.y));
            }
            if (c.stash && c.l >= 2 && dy == c.l - 1 && mk != c.mD) {
                const int p = atomicAdd(s_nst, 1);
                if (p < kLStash) {
                    S.st_p[p] = mk < c.E ? y : (y | INT32_MIN);  // high bit: already claimed
                    S.st_t[p] = (short)t;
                }
            }
            return 0.0;
    }
}

// Flattened pass over entries [e_beg, e_end) of the chunk's rows (S.off holds
// cnt + 1 exclusive offsets, S.beg the row starts).  Contributions are summed
// into c.acc[t] (or kept per entry in c.ev).  Ends with a barrier.
template <int K>
__device__ __forceinline__ void lean_pass_k(const PassCtx &c, LeanSmem &S, int *s_nst, const GView &g, int cnt,
                                            int e_beg, int e_end, uint32_t &bytes, uint32_t &scanned) {
    const int tid = threadIdx.x;
    const bool spec = e_end - e_beg <= kSpecEntries;
#ifdef DBC_LEAN_PTRACE
    long long pt = clock64();
    auto ptick = [&](int q) {
        if (K == kPUp && c.ptr && tid == 0) {
            const long long t2 = clock64();
            c.ptr[q] += (unsigned long long)(t2 - pt);
            pt = t2;
        }
    };
#else
    auto ptick = [](int) {};
#endif
    for (int base = e_beg; base < e_end; base += kBlock * kLU) {
        const int e0 = base + tid * kLU;
        int t[kLU], y[kLU], dy[kLU];
        double2 q[kLU];
        uint32_t mk[kLU];
        int cur = 0;
        if (e0 < e_end) {
            int lo = 0, hi = cnt - 1;
            while (lo < hi) {
                const int mid = (lo + hi + 1) >> 1;
                if (S.off[mid] <= e0) lo = mid; else hi = mid - 1;
            }
            cur = lo;
        }
#pragma unroll
        for (int u = 0; u < kLU; ++u) {
            const int e = e0 + u;
            t[u] = -1;
            y[u] = 0;
            if (e < e_end) {
                while (S.off[cur + 1] <= e) ++cur;
                t[u] = cur;
                y[u] = ldg_i(g.col + S.beg[cur] + (e - S.off[cur]));
            }
        }
        ptick(0);
        if (spec) {  // narrow pass (latency-bound): gather d, (sigma, delta) and the flag together
            constexpr int s = pass_spec<K>();
#pragma unroll
            for (int u = 0; u < kLU; ++u) {
                const bool on = t[u] >= 0;
                dy[u] = on ? __ldcg(c.st.d + y[u]) : kInf;
                q[u] = (on && (s & 1)) ? __ldcg(c.st.sd + y[u]) : make_double2(0.0, 0.0);
                mk[u] = (on && (s & 2)) ? __ldcg(c.mark + y[u]) : 0u;
            }
        } else {  // wide pass: the second gather only where the d test passes
#pragma unroll
            for (int u = 0; u < kLU; ++u) dy[u] = t[u] >= 0 ? __ldcg(c.st.d + y[u]) : kInf;
#pragma unroll
            for (int u = 0; u < kLU; ++u) {
                const int s = t[u] >= 0 ? pass_sel<K>(c, S, t[u], dy[u]) : 0;
                q[u] = (s & 1) ? __ldcg(c.st.sd + y[u]) : make_double2(0.0, 0.0);
                mk[u] = (s & 2) ? __ldcg(c.mark + y[u]) : 0u;
            }
        }
        ptick(1);
        bool low[kLU];
        uint32_t clm[kLU];
#pragma unroll
        for (int u = 0; u < kLU; ++u) {
            double v = 0.0;
            low[u] = false;
            clm[u] = 0u;
            if (t[u] >= 0) {
                ++scanned;
                v = pass_visit<K>(c, S, s_nst, t[u], y[u], dy[u], q[u], mk[u], bytes, &low[u], &clm[u]);
                if (c.ev) c.ev[e0 + u] = v;
            }
            if (!c.ev) acc_add(c.acc, v != 0.0 ? t[u] : -1, v);
        }
        // the requested atomics, all of this thread's entries in flight together
        if (K == kPDown) {
            int old[kLU];
#pragma unroll
            for (int u = 0; u < kLU; ++u) old[u] = low[u] ? atomicMin(c.st.d + y[u], c.l + 1) : 0;
#pragma unroll
            for (int u = 0; u < kLU; ++u)
                if (low[u] && old[u] > c.l + 1) {  // the first lowerer records the old d
                    c.lowrec[y[u]] = c.E64 | (uint32_t)old[u];
                    *c.low = 1;
                    bytes += 4;
                }
        }
        ptick(2);
        uint32_t prev[kLU];
#pragma unroll
        for (int u = 0; u < kLU; ++u) prev[u] = clm[u] ? atomicMax(c.mark + y[u], clm[u]) : 0xffffffffu;
#pragma unroll
        for (int u = 0; u < kLU; ++u)
            if (prev[u] < c.E) {  // claimed: append to the pass's list
                const int p = atomicAdd(c.ctr, 1);
                c.list[p] = y[u];
                if (c.mir && p - c.mbase < kLCap) c.mir[p - c.mbase] = y[u];
                if (c.dmir && p < kDMir) c.dmir[p] = y[u];
                if (K == kPRem) {  // removal targets keep their level
                    c.list2[p] = dy[u];
                    atomicMin(c.rmin, dy[u]);
                    atomicMax(c.rmax, dy[u]);
                }
            }
        ptick(3);
    }
    __syncthreads();
    ptick(4);
#ifdef DBC_LEAN_PTRACE
    if (K == kPUp && c.ptr && tid == 0) c.ptr[5] += 1;
#endif
}

// one specialised pass per kind (no kind switch in the entry loop)
__device__ __forceinline__ void lean_pass(const PassCtx &c, LeanSmem &S, int *s_nst, const GView &g, int cnt,
                                          int e_beg, int e_end, uint32_t &bytes, uint32_t &scanned) {
    switch (c.kind) {
        case kPDown: lean_pass_k<kPDown>(c, S, s_nst, g, cnt, e_beg, e_end, bytes, scanned); break;
        case kPUp: lean_pass_k<kPUp>(c, S, s_nst, g, cnt, e_beg, e_end, bytes, scanned); break;
        case kPRem: lean_pass_k<kPRem>(c, S, s_nst, g, cnt, e_beg, e_end, bytes, scanned); break;
        case kPDPush: lean_pass_k<kPDPush>(c, S, s_nst, g, cnt, e_beg, e_end, bytes, scanned); break;
        default: lean_pass_k<kPDRow>(c, S, s_nst, g, cnt, e_beg, e_end, bytes, scanned); break;
    }
}

// resident CTAs per SM the registers are sized for: 128 registers at 128, 256
// and 512 threads (one 512-thread CTA per SM: R-MAT 16 Mode S +9%, single-edge
// update -10% against two 64-register CTAs), 64 at 1024
#ifndef DBC_LEAN_MINB
#define DBC_LEAN_MINB (kBlock <= 128 ? 4 : (kBlock == 256 ? 2 : 1))
#endif
__global__ void __launch_bounds__(kBlock, DBC_LEAN_MINB) lean_kernel(UpdateArgs a) {
    __shared__ LeanSmem S;
    extern __shared__ double s_dyn[];  // dynamic: D list copy (old sigma, then ids, then old d)
    double *s_dsig = s_dyn;
    int *s_dmir = reinterpret_cast<int *>(s_dyn + kDMir);
    int *s_dold = s_dmir + kDMir;
    __shared__ int s_slot, s_nwork, s_dcnt, s_ucnt[2], s_rcnt, s_rmin, s_rmax, s_nst, s_nsc, s_low, s_ds;
    __shared__ int s_mirbad;  // bit (L & 1): the down mirror of level L is incomplete; bit 2 + i: up list i's
    __shared__ unsigned long long s_tph[10];  // tuning.trace_slot: SM cycles per phase of that root (thread 0)
    __shared__ int s_hb, s_hpick, s_hseq, s_hidle;

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
    int32_t *Ul[2] = {a.ws.U0 + (size_t)wk * n, a.ws.U1 + (size_t)wk * n};
    int32_t *Rv = a.ws.Rv + (size_t)wk * n;
    int32_t *Rl = a.ws.Rl + (size_t)wk * n;
    uint32_t epoch = a.ws.wepoch[wk];
    const GView &g = a.g;
    LeanBoard *board = (LeanBoard *)a.lean_board;  // nullptr: no cooperative help
    LeanBoard *mine = board ? board + wk : nullptr;
    int *live = a.next_slot + 2;                   // [0] roots finished, [1] idle workers
    const int total_roots = a.slot_list ? a.slot_count : a.k_loc;
    const bool pull = a.pull_delta != 0;  // DBC_FLAG_PULL_DELTA (no help board then)
    int hseq = 0;
    unsigned long long *stl = a.stats + kStCount + (size_t)(wk % kStLanes) * kStTraceN;  // this CTA's counter lane

    // phase clocks of one traced root (dbc_tuning.trace_slot; diagnostic): down
    // item load / scan / pass / finalize, removal, up level setup, D rows, up
    // item load / scan / pass
    bool trace = false;
    long long tclk = 0;
    if (tid == 0)
        for (int q = 0; q < 10; ++q) s_tph[q] = 0;
    // per-CTA record after the root records (dbc_debug_cta_profile): entry, end of the work loops, exit
    unsigned long long *cta_prof = a.root_prof ? a.root_prof + 6 * (size_t)max(a.k_loc, 1) + 3 * (size_t)wk : nullptr;
    if (cta_prof && tid == 0) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        cta_prof[0] = t;
    }
    auto tick = [&](int ph) {
        if (trace && tid == 0) {
            const long long t = clock64();
            if (ph >= 0) s_tph[ph] += (unsigned long long)(t - tclk);
            tclk = t;
        }
    };
    // counters: thread-local bytes / scanned entries, thread 0's tallies
    uint32_t my_bytes = 0, my_scan = 0;
    uint32_t sc_ph[6] = {0, 0, 0, 0, 0, 0};  // scanned: down, removal, D rows, level-2 probes, up@2, up@>=3
    unsigned long long c_case[3] = {0, 0, 0}, c_touch = 0, c_down = 0, c_lev[2] = {0, 0};

    // Run a pass over the chunk in S (cnt rows, Etot entries): locally, or
    // published on the board when it is wide and idle workers exist.  c holds
    // the local (shared-memory) counters; they are updated either way.
    // Returns bit 0: the per-row sums are in S.acc (else in S.ev, per entry);
    // bit 1: the pass was published (helped).
    auto run_pass = [&](PassCtx c, int cnt, int Etot, int slot, int sel, uint32_t &scan) -> int {
        const int nblk = (Etot + kHelpBlk - 1) / kHelpBlk;
        if (nblk >= kHelpMinBlk) {
            if (tid == 0) s_hidle = mine ? __ldcg(live + 1) : 0;
            __syncthreads();
        }
        if (nblk < kHelpMinBlk || s_hidle <= 0) {
            c.ev = Etot <= kLEnt ? S.ev : nullptr;
            lean_pass(c, S, &s_nst, g, cnt, 0, Etot, my_bytes, scan);
            return c.ev == nullptr ? 1 : 0;
        }
        // publish: chunk mirror + context (visible device-wide), then the word
        for (int t = tid; t < cnt; t += kBlock) {
            mine->off[t + 1] = S.off[t + 1];
            mine->beg[t] = S.beg[t];
            mine->aux[t] = S.aux[t];
            mine->c0[t] = S.c0[t];
            mine->c1[t] = S.c1[t];
            mine->v[t] = S.v[t];
            mine->acc[t] = 0.0;
        }
        __threadfence();
        __syncthreads();
        if (tid == 0) {
            mine->off[0] = 0;
            mine->done = 0;
            mine->ctr = *c.ctr;
            mine->low = 0;
            mine->rmin = c.rmin ? *c.rmin : 0;
            mine->rmax = c.rmax ? *c.rmax : 0;
            mine->kind = c.kind;
            mine->slot = slot;
            mine->l = c.l;
            mine->cnt = cnt;
            mine->Etot = Etot;
            mine->sel = sel;
            mine->E = c.E;
            mine->epoch = (uint32_t)(c.E64 >> 32);
            mine->ul = c.ul;
            mine->uh = c.uh;
            mine->pull = c.pull ? 1 : 0;
            hseq = (hseq + 1) & 0xFFFF;
            __threadfence();
            atomicExch(&mine->word, hb_pack(1, nblk, 0, hseq));
            atomicAdd(a.next_slot + 1, 1);  // open requests (idle workers poll this word only)
            atomicAdd(stl + kStHelpReq, 1ull);
            atomicAdd(stl + kStHelpBlkAll, (unsigned long long)nblk);
        }
        PassCtx gc = c;
        gc.ctr = &mine->ctr;
        gc.low = &mine->low;
        gc.rmin = &mine->rmin;
        gc.rmax = &mine->rmax;
        gc.acc = mine->acc;
        gc.ev = nullptr;
        gc.stash = false;  // helpers' shared memory is their own: D-row pushes run as a kPDPush pass
        gc.mir = nullptr;  // helpers append to the list only: its mirror is incomplete
        gc.dmir = nullptr;
        if (tid == 0 && c.mir) s_mirbad |= c.mirbit;
        if (tid == 0 && c.dmir) s_mirbad |= 256;  // the D id mirror too
        for (;;) {  // the owner takes blocks too
            if (tid == 0) {
                const unsigned long long w = atomicAdd(&mine->word, 1ull << 16);
                s_hb = hb_next(w) < nblk ? hb_next(w) : -1;
            }
            __syncthreads();
            const int b = s_hb;
            __syncthreads();
            if (b < 0) break;
            lean_pass(gc, S, &s_nst, g, cnt, b * kHelpBlk, min(Etot, (b + 1) * kHelpBlk), my_bytes, scan);
            if (tid == 0) {
                __threadfence();
                atomicAdd(&mine->done, 1);
            }
        }
        if (tid == 0) {
            while (atomicAdd(&mine->done, 0) < nblk) __nanosleep(200);
            atomicExch(&mine->word, hb_pack(0, 0, 0, hseq));
            atomicSub(a.next_slot + 1, 1);
            __threadfence();
            *c.ctr = __ldcg(&mine->ctr);
            if (__ldcg(&mine->low)) *c.low = 1;
            if (c.rmin) *c.rmin = __ldcg(&mine->rmin);
            if (c.rmax) *c.rmax = __ldcg(&mine->rmax);
        }
        __syncthreads();
        for (int t = tid; t < cnt; t += kBlock) S.acc[t] = __ldcg(mine->acc + t);
        __syncthreads();
        return 3;
    };

    for (;;) {
        if (tid == 0) {
            const int slot = atomicAdd(a.next_slot, 1);
            s_slot = slot < total_roots ? (a.slot_list ? a.slot_list[slot] : slot) : -1;
        }
        __syncthreads();
        const int slot = s_slot;
        __syncthreads();
        if (slot < 0) break;
        const Root st{a.d + (size_t)slot * n, a.sd + (size_t)slot * n};
        const int sroot = a.roots[slot];
        trace = slot == a.trace_slot;
        bool masks_dropped = false;
        // root profile (dbc_debug_root_profile): start, jobs, touched, levels (thread 0)
        unsigned long long pr_t0 = 0, pr_jobs = 0, pr_touch = c_touch, pr_lev = c_lev[0] + c_lev[1];
        if (a.root_prof && tid == 0) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(pr_t0));

        for (int w0 = a.ins_begin; w0 < a.ins_end;) {
            // ---- classification (K2) of a window of insertions, in parallel ----
            const int nw = min(kLWin, a.ins_end - w0);
            bool work = false;
            if (tid < nw) {  // (kLWin <= kBlock)
                const int u = __ldg(a.ins_u + w0 + tid), v = __ldg(a.ins_v + w0 + tid);
                const int du = __ldcg(st.d + u), dv = __ldcg(st.d + v);
                work = du != dv;
                S.wul[tid] = du < dv ? v : u;
                S.wlev[tid] = work ? min(du, dv) + 1 : INT32_MAX;
                my_bytes += 8;
            }
            {  // ordered list of the working insertions of the window
                const int rank = block_excl_scan(work ? 1 : 0, &s_nwork);
                if (work) S.wq[rank] = tid;
            }
            __syncthreads();
            const int nwork = s_nwork;
            int next = nw;  // window positions consumed (a Case-3 job stops the window after it)
            for (int qi = 0; qi < nwork; ++qi) {
                const int q = S.wq[qi];
                const int ins = w0 + q;
                const int ul = S.wul[q], L0 = S.wlev[q];
                const int uh = (__ldg(a.ins_u + ins) == ul) ? __ldg(a.ins_v + ins) : __ldg(a.ins_u + ins);
                const int lim = ins;
                ++epoch;
                const uint32_t E = epoch << 2, mD = E | kLD, mU = E | kLUp;
                const unsigned long long E64 = (unsigned long long)epoch << 32;
                if (!masks_dropped) {  // update.cu's level-2 masks are not maintained here
                    if (tid == 0 && a.mask_ds[slot] >= 0) a.mask_ds[slot] = -1;
                    masks_dropped = true;
                }
                PassCtx pc;
                pc.E = E;
                pc.mD = mD;
                pc.mU = mU;
                pc.E64 = E64;
                pc.st = st;
                pc.mark = mark;
                pc.lowrec = lowrec;
                pc.dacc = dacc;
                pc.low = &s_low;
                pc.rmin = &s_rmin;
                pc.rmax = &s_rmax;
                pc.acc = S.acc;
                pc.ev = nullptr;
                pc.full = a.scen != nullptr || pull;
                pc.pull = pull;
                pc.ul = ul;
                pc.uh = uh;
                pc.stash = false;
                pc.ptr = trace ? a.stats + kStTrace0 : nullptr;
                pc.mir = nullptr;
                pc.dmir = nullptr;
                pc.mbase = 0;
                pc.mirbit = 0;
                // ---- seed (A2) ----
                if (tid == 0) {
                    const int dl = __ldcg(st.d + ul);
                    const bool c3 = dl > L0;
                    if (c3) {
                        st.d[ul] = L0;
                        lowrec[ul] = E64 | (uint32_t)dl;
                        ++c_case[2];
                    } else {
                        ++c_case[1];
                    }
                    s_low = c3;
                    mark[ul] = mD;
                    Dv[0] = ul;
                    s_dmir[0] = ul;
                    S.nx[0] = ul;
                    s_mirbad = 0;
                    Doff[0] = 0;
                    Doff[1] = 1;
                    s_dcnt = 1;
                    s_ucnt[0] = s_ucnt[1] = 0;
                    s_rcnt = 0;
                    s_rmin = INT32_MAX;
                    s_rmax = 0;
                    my_bytes += 4 + (c3 ? 12 : 0);
                }
                __syncthreads();

                // ---- down phase (K3) ----
                int L = L0, lb = 0, le = 1, nlev = 0;
                tick(-1);
                while (lb < le) {
                    // the first kLCap vertices of this level come from the shared
                    // mirror its producer pass filled (unless helpers appended)
                    const bool mir_ok = !(s_mirbad & (1 << (L & 1)));
                    for (int c = lb; c < le; c += kLCap) {
                        const int cnt = min(kLCap, le - c);
                        if (c == lb && tid == 0) s_mirbad &= ~(1 << ((L + 1) & 1));  // the next level's
                        for (int t = tid; t < cnt; t += kBlock) {
                            const int w = (c == lb && mir_ok) ? S.nx[t] : __ldcg(Dv + c + t);
                            const int2 r = row_of(g, w, lim);
                            const unsigned long long lr = __ldcg(lowrec + w);
                            const int od = ((lr >> 32) == epoch) ? (int)(uint32_t)lr : L;
                            const double os = __ldcg(&st.sd[w].x);
                            Dold[c + t] = od;
                            Dsig[c + t] = os;
                            if (c + t < kDMir) {
                                s_dold[c + t] = od;
                                s_dsig[c + t] = os;
                            }
                            S.v[t] = w;
                            S.beg[t] = r.x;
                            S.off[t + 1] = r.y - r.x;
                            S.acc[t] = 0.0;
                            my_bytes += 8 + 20;
                        }
                        __syncthreads();
                        tick(0);
                        const int Etot = chunk_offsets(S, cnt);
                        tick(1);
                        PassCtx cdn = pc;
                        cdn.kind = kPDown;
                        cdn.l = L;
                        cdn.list = Dv;
                        cdn.ctr = &s_dcnt;
                        cdn.mir = S.nx;
                        cdn.dmir = s_dmir;
                        cdn.mbase = le;
                        cdn.mirbit = 1 << ((L + 1) & 1);
                        const bool in_acc = run_pass(cdn, cnt, Etot, slot, 0, sc_ph[0]) & 1;
                        for (int t = tid; t < cnt; t += kBlock) {
                            double sum;
                            const int w = S.v[t];
                            if (!in_acc) {  // canonical order: the row's entries left to right
                                sum = 0.0;
                                for (int e = S.off[t]; e < S.off[t + 1]; ++e) sum = __dadd_rn(sum, S.ev[e]);
                            } else if ((sum = S.acc[t]) >= kExact) {  // order matters above 2^53: re-sum
                                const int2 r = row_of(g, w, lim);
                                sum = 0.0;
                                for (int j = r.x; j < r.y; ++j) {
                                    const int x = ldg_i(g.col + j);
                                    if (__ldcg(st.d + x) == L - 1) sum = __dadd_rn(sum, __ldcg(&st.sd[x].x));
                                }
                            }
                            st.sd[w].x = sum;
                            my_bytes += 8;
                            if (!(sum <= 1.7976931348623157e308)) atomicOr(a.err, kErrNumeric);
                        }
                        __syncthreads();
                    }
                    tick(2);
                    lb = le;
                    le = s_dcnt;
                    ++nlev;
                    ++L;
                    if (tid == 0) Doff[nlev + 1] = le;
                }
                const int Lmax = L - 1;  // deepest D level
                const int dtotal = le;
                const bool dmir_ok = !(s_mirbad & 256);  // the D id copy is complete (no helped down pass)

                // ---- removal pushes (A4 step 0, Case 3) ----
                if (s_low) {
                    for (int c = 0; c < dtotal; c += kLCap) {
                        const int cnt = min(kLCap, dtotal - c);
                        for (int t = tid; t < cnt; t += kBlock) {
                            const int j = c + t;
                            const int w = (j < kDMir && dmir_ok) ? s_dmir[j] : __ldcg(Dv + j);
                            const int od = j < kDMir ? s_dold[j] : __ldcg(Dold + j);
                            const int dw = __ldcg(st.d + w);
                            int len = 0;
                            if (od != dw && od != kInf) {
                                const int2 r = row_of(g, w, lim);
                                len = r.y - r.x;
                                S.beg[t] = r.x;
                                const double dold = __ldcg(&st.sd[w].y);  // delta is still the old one
                                S.c0[t] = -__ddiv_rn(__dadd_rn(1.0, dold), j < kDMir ? s_dsig[j] : __ldcg(Dsig + j));
                                S.aux[t] = od - 1;
                                my_bytes += 8 + 16;
                            }
                            S.v[t] = w;
                            S.off[t + 1] = len;
                        }
                        __syncthreads();
                        const int Etot = chunk_offsets(S, cnt);
                        PassCtx cr = pc;
                        cr.kind = kPRem;
                        cr.l = 0;
                        cr.list = Rv;
                        cr.list2 = Rl;
                        cr.ctr = &s_rcnt;
                        run_pass(cr, cnt, Etot, slot, 0, sc_ph[1]);
                    }
                }
                __syncthreads();

                tick(4);
                // ---- up phase (K4 + Alg. 8) ----
                const int rcnt = s_rcnt, rmin = s_rmin, rmax = s_rmax;
                int cu = 0;  // Ul[cu] holds the up vertices of the current level
                int nup = 0;
                if (tid == 0) s_ds = -1;
                for (int l = max(Lmax, rcnt ? rmax : 0); l >= 1; --l) {
                    // removal targets of this level join the up list
                    if (rcnt && l >= rmin && l <= rmax) {
                        for (int j = tid; j < rcnt; j += kBlock)
                            if (__ldcg(Rl + j) == l) {
                                const int p = atomicAdd(&s_ucnt[cu], 1), x = __ldcg(Rv + j);
                                Ul[cu][p] = x;
                                if (p < kLCap) S.um[cu][p] = x;
                            }
                    }
                    if (l == 2 && tid == 0) {  // the root's row: level-1 candidates of the shortcut
                        const int2 rs = row_of(g, sroot, lim);
                        s_ds = rs.y - rs.x <= kLAdj ? rs.y - rs.x : -1;
                    }
                    if (tid == 0) s_mirbad &= ~(4 << (cu ^ 1));  // the list this level produces
                    __syncthreads();
                    const bool umir_ok = !(s_mirbad & (4 << cu));  // its shared mirror is complete
                    tick(5);
                    if (l == 2 && s_ds > 0) {
                        const int2 rs = row_of(g, sroot, lim);
                        for (int j = tid; j < s_ds; j += kBlock) S.adjs[j] = ldg_i(g.col + rs.x + j);
                    }
                    const int nd = (l >= L0 && l <= Lmax) ? Doff[l - L0 + 1] - Doff[l - L0] : 0;
                    const int db = (l >= L0 && l <= Lmax) ? Doff[l - L0] : 0;
                    const int nu = s_ucnt[cu];
                    const int ds = s_ds;
                    PassCtx cp = pc;
                    cp.l = l;
                    cp.list = Ul[cu ^ 1];
                    cp.ctr = &s_ucnt[cu ^ 1];
                    cp.mir = S.um[cu ^ 1];
                    cp.mbase = 0;
                    cp.mirbit = 4 << (cu ^ 1);
                    // D vertices of the level: delta by pull, pushes to predecessors
                    // outside D.  DBC_FLAG_PULL_DELTA: the up vertices too (rows
                    // nd.. of this loop, aux = -1): every touched vertex pulls
                    // delta in canonical order, predecessors are only claimed.
                    const int npull = nd + (pull ? nu : 0);
                    for (int c = 0; c < npull; c += kLCap) {
                        const int cnt = min(kLCap, npull - c);
                        if (tid == 0) s_nst = 0;
                        for (int t = tid; t < cnt; t += kBlock) {
                            const int j = c + t;
                            const int x = j < nd ? ((db + j < kDMir && dmir_ok) ? s_dmir[db + j] : __ldcg(Dv + db + j))
                                          : ((j - nd < kLCap && umir_ok) ? S.um[cu][j - nd] : __ldcg(Ul[cu] + j - nd));
                            const double2 q = __ldcg(st.sd + x);  // (sigma_new, delta_old)
                            const int2 r = row_of(g, x, lim);
                            S.v[t] = x;
                            S.beg[t] = r.x;
                            S.aux[t] = j < nd ? db + j : -1;
                            S.c0[t] = q.x;
                            S.c1[t] = q.y;
                            S.off[t + 1] = r.y - r.x;
                            S.acc[t] = 0.0;
                            my_bytes += 8 + 16;
                        }
                        __syncthreads();
                        const int Etot = chunk_offsets(S, cnt);
                        PassCtx cd = cp;
                        cd.kind = kPDRow;
                        cd.stash = true;
                        const int how = run_pass(cd, cnt, Etot, slot, cu ^ 1, sc_ph[2]);
                        const bool in_acc = how & 1, helped = how & 2;
                        for (int t = tid; t < cnt; t += kBlock) {  // delta, BC, the push coefficients
                            const int x = S.v[t], di = S.aux[t];
                            double dn = S.acc[t];
                            if (!in_acc) {  // Eq. (2) summed left to right in canonical order
                                dn = 0.0;
                                for (int e = S.off[t]; e < S.off[t + 1]; ++e) dn = __dadd_rn(dn, S.ev[e]);
                            } else if (pull) {  // a chunk too wide for the entry buffer: re-sum in order
                                const int2 r = row_of(g, x, lim);
                                dn = 0.0;
                                for (int e = r.x; e < r.y; ++e) {
                                    const int y = ldg_i(g.col + e);
                                    if (__ldcg(st.d + y) != l + 1) continue;
                                    const double2 qy = __ldcg(st.sd + y);
                                    dn = __dadd_rn(dn, __dmul_rn(__ddiv_rn(S.c0[t], qy.x), __dadd_rn(1.0, qy.y)));
                                }
                            }
                            const double sn = S.c0[t], dold = S.c1[t];
                            if (dn != dold) {
                                atomicAdd(a.bc + x, __dsub_rn(dn, dold));
                                st.sd[x].y = dn;
                            }
                            if (di >= 0) {
                                const bool lowered = (di < kDMir ? s_dold[di] : __ldcg(Dold + di)) != l;
                                S.c0[t] = __ddiv_rn(__dadd_rn(1.0, dn), sn);
                                S.c1[t] = lowered ? 0.0 : __ddiv_rn(__dadd_rn(1.0, dold), di < kDMir ? s_dsig[di] : __ldcg(Dsig + di));
                            }
                            my_bytes += 16 + 16;
                        }
                        __syncthreads();
                        const int nst = s_nst;
                        if (!helped && nst <= kLStash) {  // the staged predecessors
                            for (int j = tid; j < nst; j += kBlock) {
                                const int t = S.st_t[j], pr = S.st_p[j], p = pr & INT32_MAX;
                                if (pull) {  // the predecessor pulls its own delta at level l - 1
                                    if (pr >= 0) claim_append(cp, p, mU);
                                    continue;
                                }
                                const bool new_edge = S.v[t] == ul && p == uh;
                                const double w = new_edge ? S.c0[t] : __dsub_rn(S.c0[t], S.c1[t]);
                                if (w != 0.0) atomicAdd(dacc + p, w);
                                my_bytes += 16;
                                if ((w != 0.0 || cp.full) && pr >= 0) claim_append(cp, p, mU);
                            }
                        } else {  // stash overflow, or a helped pull: a push pass over the rows
                            PassCtx cpu = cp;
                            cpu.kind = kPDPush;
                            run_pass(cpu, cnt, Etot, slot, cu ^ 1, sc_ph[3]);
                        }
                        __syncthreads();
                    }
                    tick(6);
                    // up vertices of the level: apply Ddelta, forward it to the predecessors
                    for (int c = 0; c < (pull ? 0 : nu); c += kLCap) {
                        const int cnt = min(kLCap, nu - c);
                        if (tid == 0) s_nsc = 0;
                        __syncthreads();
                        for (int t = tid; t < cnt; t += kBlock) {
                            const int x = (c + t < kLCap && umir_ok) ? S.um[cu][c + t] : __ldcg(Ul[cu] + c + t);
                            // the row bounds are loaded with the accumulator (one round trip)
                            const int rb0 = ldg_i(g.rp + x), re0 = ldg_i(g.rp + x + 1);
                            const double f = __ldcg(dacc + x);
                            const double2 q = __ldcg(st.sd + x);
                            const double gd = __dmul_rn(q.x, f);
                            dacc[x] = 0.0;
                            if (gd != 0.0) {
                                st.sd[x].y = __dadd_rn(q.y, gd);
                                atomicAdd(a.bc + x, gd);
                            }
                            my_bytes += 40;
                            S.v[t] = x;
                            S.c0[t] = f;
                            int len = 0;
                            if (l >= 2 && (f != 0.0 || cp.full)) {
                                const int2 r = rb0 >= 0 ? make_int2(rb0, re0 & kMask) : row_of(g, x, lim);
                                if (l == 2 && ds > 0 && r.y - r.x > a.short_mult * ds) {
                                    S.sc_t[atomicAdd(&s_nsc, 1)] = t;  // level-1 predecessors = adj(s) n adj(x)
                                } else {
                                    len = r.y - r.x;
                                    S.beg[t] = r.x;
                                    my_bytes += 8;
                                }
                            }
                            S.off[t + 1] = len;
                        }
                        __syncthreads();
                        tick(7);
                        const int Etot = chunk_offsets(S, cnt);
                        tick(8);
                        PassCtx cu2 = cp;
                        cu2.kind = kPUp;
                        run_pass(cu2, cnt, Etot, slot, cu ^ 1, sc_ph[l == 2 ? 4 : 5]);
                        tick(9);
                        const int nsc = s_nsc;
                        if (nsc) {
                            const int pairs = nsc * ds;
                            for (int j = tid; j < pairs; j += kBlock) {
                                const int t = S.sc_t[j / ds], p = S.adjs[j % ds];
                                my_bytes += 32;
                                ++sc_ph[3];
                                if (adjacent_visible(g, S.v[t], p, lim)) {
                                    const double f = S.c0[t];
                                    if (f != 0.0) atomicAdd(dacc + p, f);
                                    my_bytes += 16;
                                    claim_append(cp, p, mU);
                                }
                            }
                        }
                        __syncthreads();
                    }
                    nup += nu;
                    if (tid == 0) s_ucnt[cu] = 0;
                    cu ^= 1;
                    ++c_lev[1];
                    __syncthreads();
                    tick(3);
                }
                c_lev[0] += nlev;
                c_down += dtotal;
                c_touch += dtotal + nup;
                ++pr_jobs;
                if (a.scen && tid == 0)  // Fig. 2 / Fig. 4 record: case | touched << 2 | |D| << 33
                    a.scen[(size_t)ins * a.k_loc + slot] =
                        (long long)(((unsigned long long)dtotal << 33) | ((unsigned long long)(dtotal + nup) << 2) |
                                    (s_low ? 3u : 2u));
                const bool lowered_any = s_low;  // Case 3 (only Case 3 lowers distances)
                __syncthreads();
                if (lowered_any) {  // distances changed: the rest of the window is classified again
                    next = q + 1;
                    break;
                }
            }
            if (tid < next && !work) {  // Case-1 insertions consumed from this window
                ++c_case[0];
                if (a.scen) a.scen[(size_t)(w0 + tid) * a.k_loc + slot] = 1;
            }
            w0 += next;
            __syncthreads();
        }
        if (tid == 0) atomicAdd(live, 1);  // one more root finished
        if (a.root_prof) {  // per-slot record: {t0, t1, working jobs, touched, scanned (thread 0 only), levels}
            unsigned long long *rp6 = a.root_prof + 6 * (size_t)slot;
            if (tid == 0) {
                unsigned long long t1;
                asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
                rp6[0] = pr_t0;
                rp6[1] = t1;
                rp6[2] = pr_jobs;
                rp6[3] = c_touch - pr_touch;
                rp6[5] = c_lev[0] + c_lev[1] - pr_lev;
            }
        }
    }

    // ---- out of roots: take blocks of the wide passes of workers still running ----
    if (board) {
        if (tid == 0) atomicAdd(live + 1, 1);
        int cur_owner = -1, cur_seq = -1;
        const int nwk = gridDim.x;
        int backoff = 64;
        for (;;) {
            if (tid == 0) {  // wait for an open request (or the end of every root chain)
                s_hpick = 0;
                for (;;) {
                    if (__ldcg(a.next_slot + 1) > 0) break;
                    if (__ldcg(live) >= total_roots) {
                        s_hpick = -2;
                        break;
                    }
                    __nanosleep(backoff);
                    backoff = min(backoff * 2, 512);
                }
            }
            __syncthreads();
            if (s_hpick == -2) break;
            __syncthreads();
            backoff = 64;
            for (int i = tid; i < nwk; i += kBlock) {
                const int o = (wk + 1 + i) % nwk;
                const unsigned long long w = __ldcg(&board[o].word);
                const int left = hb_nblk(w) - hb_next(w);
                if (hb_open(w) && left > 0)
                    atomicMax(&s_hpick, (min(left, 0x7FFFF) << 12) | min(i, 0xFFF) | 0);
            }
            __syncthreads();
            if (tid == 0) {
                int pick = -1, b = -1, sq = -1;
                if (s_hpick != 0) {
                    pick = (wk + 1 + (s_hpick & 0xFFF)) % nwk;
                    const unsigned long long w = atomicAdd(&board[pick].word, 1ull << 16);
                    if (hb_open(w) && hb_next(w) < hb_nblk(w)) {
                        b = hb_next(w);
                        sq = hb_seq(w);
                    }
                } else if (__ldcg(live) >= total_roots) {
                    pick = -2;
                }
                s_hpick = pick;
                s_hb = b;
                s_hseq = sq;
            }
            __syncthreads();
            const int pick = s_hpick, b = s_hb, sq = s_hseq;
            __syncthreads();
            if (pick == -2) break;
            if (b < 0) {
                if (tid == 0) __nanosleep(256);
                continue;
            }
            LeanBoard *ob = board + pick;
            const int cnt = __ldcg(&ob->cnt), Etot = __ldcg(&ob->Etot);
            if (pick != cur_owner || sq != cur_seq) {  // a new request: load its chunk
                for (int t = tid; t <= cnt; t += kBlock) {
                    S.off[t] = __ldcg(ob->off + t);
                    if (t < cnt) {
                        S.beg[t] = __ldcg(ob->beg + t);
                        S.aux[t] = __ldcg(ob->aux + t);
                        S.c0[t] = __ldcg(ob->c0 + t);
                        S.c1[t] = __ldcg(ob->c1 + t);
                        S.v[t] = __ldcg(ob->v + t);
                    }
                }
                cur_owner = pick;
                cur_seq = sq;
                __syncthreads();
            }
            PassCtx c;
            c.kind = __ldcg(&ob->kind);
            c.l = __ldcg(&ob->l);
            c.E = __ldcg(&ob->E);
            c.mD = c.E | kLD;
            c.mU = c.E | kLUp;
            c.E64 = (unsigned long long)__ldcg(&ob->epoch) << 32;
            const int oslot = __ldcg(&ob->slot);
            c.st = Root{a.d + (size_t)oslot * n, a.sd + (size_t)oslot * n};
            c.mark = a.ws.mark + (size_t)pick * n;
            c.lowrec = a.ws.lowrec + (size_t)pick * n;
            c.dacc = a.ws.dacc + (size_t)pick * n;
            c.list = c.kind == kPDown ? a.ws.Dv + (size_t)pick * n
                     : c.kind == kPRem ? a.ws.Rv + (size_t)pick * n
                                       : ((__ldcg(&ob->sel) ? a.ws.U1 : a.ws.U0) + (size_t)pick * n);
            c.list2 = a.ws.Rl + (size_t)pick * n;
            c.ctr = &ob->ctr;
            c.low = &ob->low;
            c.rmin = &ob->rmin;
            c.rmax = &ob->rmax;
            c.acc = ob->acc;
            c.ev = nullptr;
            c.full = a.scen != nullptr;
            c.ul = __ldcg(&ob->ul);
            c.uh = __ldcg(&ob->uh);
            c.pull = __ldcg(&ob->pull) != 0;
            c.stash = false;
            c.ptr = nullptr;
            c.mir = nullptr;
            c.dmir = nullptr;
            uint32_t hscan = 0;
            lean_pass(c, S, &s_nst, g, cnt, b * kHelpBlk, min(Etot, (b + 1) * kHelpBlk), my_bytes, hscan);
            my_scan += hscan;
            if (tid == 0) {
                __threadfence();
                atomicAdd(&ob->done, 1);
                atomicAdd(stl + kStHelpBlk, 1ull);
            }
        }
    }

    if (cta_prof && tid == 0) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        cta_prof[1] = t;
    }
    if (tid == 0) {
        for (int q = 0; q < 10; ++q)
            if (s_tph[q]) atomicAdd(stl + kStTime0 + q, s_tph[q]);
        a.ws.wepoch[wk] = epoch;
        if (c_case[1]) atomicAdd(stl + kStCase2, c_case[1]);
        if (c_case[2]) atomicAdd(stl + kStCase3, c_case[2]);
        if (c_touch) atomicAdd(stl + kStTouched, c_touch);
        if (c_down) atomicAdd(stl + kStDown, c_down);
        if (c_lev[0]) atomicAdd(stl + kStLevDown, c_lev[0]);
        if (c_lev[1]) atomicAdd(stl + kStLevUp, c_lev[1]);
    }
    unsigned long long sc_all = 0;
#pragma unroll
    for (int q = 0; q < 6; ++q) {
        sc_all += sc_ph[q];
        if (sc_ph[q]) atomicAdd(stl + kStPhase0 + q, (unsigned long long)sc_ph[q]);
    }
    sc_all += my_scan;
    unsigned long long c1 = c_case[0], by = my_bytes;
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        c1 += __shfl_xor_sync(kFull, c1, o);
        by += __shfl_xor_sync(kFull, by, o);
        sc_all += __shfl_xor_sync(kFull, sc_all, o);
    }
    __shared__ unsigned long long s_red[3];
    if (tid < 3) s_red[tid] = 0;
    __syncthreads();
    if ((tid & 31) == 0) {
        if (c1) atomicAdd(s_red + 0, c1);
        if (by) atomicAdd(s_red + 1, by);
        if (sc_all) atomicAdd(s_red + 2, sc_all);
    }
    __syncthreads();
    if (tid == 0) {
        if (s_red[0]) atomicAdd(stl + kStCase1, s_red[0]);
        if (s_red[1]) atomicAdd(stl + kStBytes, s_red[1]);
        if (s_red[2]) atomicAdd(stl + kStScanned, s_red[2]);
    }
    if (tid == 0) {  // the last CTA out zeroes the launch counters for the next launch (no memset)
        __threadfence();
        if (atomicAdd(a.next_slot + 4, 1) == (int)gridDim.x - 1) {
            for (int q = 0; q < 5; ++q) a.next_slot[q] = 0;
            __threadfence();
        }
    }
    if (cta_prof && tid == 0) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        cta_prof[2] = t;
    }
}

}  // namespace

#if DBC_BLOCK == 128
size_t lean_board_bytes() { return sizeof(LeanBoard); }
#endif

#define DBC_CAT2(a, b) a##b
#define DBC_CAT(a, b) DBC_CAT2(a, b)
#ifndef DBC_LEAN_SUFFIX
#define DBC_LEAN_SUFFIX DBC_BLOCK
#endif
void DBC_CAT(launch_update_lean_, DBC_LEAN_SUFFIX)(const UpdateArgs &a, int workers, cudaStream_t s) {
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(lean_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kLDyn);
        attr = true;
    }
    lean_kernel<<<workers, kBlock, kLDyn, s>>>(a);
}

int DBC_CAT(lean_resident_, DBC_LEAN_SUFFIX)() {
    int nb = 0;
    cudaFuncSetAttribute(lean_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kLDyn);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, lean_kernel, kBlock, kLDyn);
    return nb;
}

}  // namespace dbc
