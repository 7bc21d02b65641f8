// dbc_internal.cuh -- shared device-side definitions of libdbc (B200 / sm_100a).
//
// Layout in HBM:
//   graph   rp int32[n+1] (bit 31 of rp[v] = "row v has entries of the current
//           batch"), col int32[cap] in canonical order, scol int32[cap] (same
//           rows sorted by id); for flagged rows xinfo[v] = {first, count} into
//           the batch arrays xtag (insertion index) / xnbr (neighbour).  Row v at
//           insertion i = base part + batch entries with index <= i.
//   state   root-major (each root's arrays contiguous): d int32[k_loc][n], the
//           filter every neighbour gather reads (kept apart from sigma/delta so
//           the filter footprint stays small and L2-friendly), and sd
//           double2[k_loc][n] = (sigma, delta), so the successor pair of Eq. (2)
//           arrives in one 16-byte gather; bc double[n].
//   scratch per persistent worker CTA, n-sized arrays (epoch-tagged, never
//           cleared between jobs -- no O(n) work per root per insertion,
//           SURVEY.md Sec. 7 hard part (iii)).
#pragma once

#include <cstdint>
#include <type_traits>

#include <cuda_runtime.h>

namespace dbc {

// threads per worker CTA; the kernels are compiled once per value (Makefile):
// 256 (2 CTAs/SM) for few roots with hub-heavy rows, 128 (4 CTAs/SM) when
// there are more roots than 2 x #SMs (all root chains resident at once).
#ifndef DBC_BLOCK
#define DBC_BLOCK 256
#endif
// resident CTAs per SM the register budget is sized for (__launch_bounds__)
#if DBC_BLOCK == 512 && defined(DBC_MINB512)
#define DBC_MINB DBC_MINB512
#elif DBC_BLOCK == 256 && defined(DBC_MINB256)
#define DBC_MINB DBC_MINB256
#endif
#ifndef DBC_MINB
#define DBC_MINB ((512 / DBC_BLOCK) > 0 ? (512 / DBC_BLOCK) : 1)
#endif
constexpr int kBlock = DBC_BLOCK;
constexpr int kMinBlocks = DBC_MINB;
constexpr int kWarps = kBlock / 32;
constexpr int kSmallDeg = 32;            // rows <= this are walked by one lane
constexpr uint32_t kFull = 0xffffffffu;
constexpr int32_t kInf = INT32_MAX;
constexpr int32_t kMask = 0x7fffffff;
constexpr uint32_t kDown = 1u;           // mark state: in the down set D (Alg. 2 t[v] = down)
constexpr uint32_t kUp = 2u;             // mark state: queued by the up phase (t[v] = up)
constexpr uint32_t kUpDone = 3u;         // mark state: up vertex processed
constexpr double kExact = 9007199254740992.0;  // 2^53

enum ErrBits : int { kErrNumeric = 1, kErrOverflow = 2 };

// Counters accumulated by the kernels (device, u64).
enum StatIdx : int {
    kStCase1 = 0, kStCase2, kStCase3, kStTouched, kStDown, kStScanned, kStBytes,
    kStStaticBytes,
    kStPhase0,                 // 6: entries scanned by down / removal / D-pull / D-push / up@2 / up@>=3
    kStTime0 = kStPhase0 + 6,  // 10 timers (ns, thread 0), see update.cu tick()
    kStLevDown = kStTime0 + 10,  // level steps of the down phase
    kStLevUp,                    // level steps of the up phase
    kStHelpReq,                  // C2 passes published for cooperative help
    kStHelpBlk,                  // blocks of them processed by helpers
    kStHelpBlkAll,               // all blocks of published passes
    kStGroups,                   // Case-2 group jobs (>= 2 insertions repaired together)
    kStGroupIns,                 // insertions in those group jobs
    kStBusyBlk,                  // help blocks run by busy workers (at their level boundaries)
    kStDeferred,                 // long rows of wide up levels processed in deferred chunks
    kStUpPass,                   // in-lane passes of wide up levels published as help blocks (kind 5)
    kStTraceN,                   // -DDBC_PHASE_TIMERS: events of the traced slot (DBC_TRACE_SLOT)
    kStTrace0,                   // kTraceCap (code, %globaltimer) pairs
    kStCount = kStTrace0 + 2 * 1024
};
constexpr int kTraceCap = 1024;
// Contention-free copies of the counters below kStTraceN: kernels whose CTAs
// all finish together (the per-insertion kernel) add into lane (CTA % kStLanes)
// at stats + kStCount + lane * kStTraceN; read_stats folds the lanes in.
constexpr int kStLanes = 64;
constexpr int kStAlloc = kStCount + kStLanes * kStTraceN;
__device__ __forceinline__ unsigned long long *stat_lane(unsigned long long *stats) {
    return stats + kStCount + (size_t)(blockIdx.x % kStLanes) * kStTraceN;
}
// Sum of v over the warp added to counter idx of the CTA's lane (all 32 lanes must call).
__device__ __forceinline__ void stat_add_warp(unsigned long long *stats, int idx, unsigned long long v) {
#pragma unroll
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((threadIdx.x & 31) == 0 && v) atomicAdd(stat_lane(stats) + idx, v);
}

// The state of one root (pointers into the root-major arrays).
struct Root {
    int32_t *d;    // distance, kInf = unreachable
    double2 *sd;   // (sigma, delta)
    __device__ __forceinline__ int dist(int y) const { return d[y]; }
};

struct GView {
    const int32_t *__restrict__ rp;
    const int32_t *__restrict__ col;   // rows in canonical order
    const int32_t *__restrict__ scol;  // the same rows sorted by neighbour id
    const int2 *__restrict__ xinfo;
    const int32_t *__restrict__ xtag;
    const int32_t *__restrict__ xnbr;  // neighbour of each batch entry (parallel to xtag)
};

// Scratch of the persistent workers (one CTA = one worker), each array
// worker-major with stride n.
// A resolved long row of a wide up level waiting for a later chunk (down rows
// from the front of the per-worker array, up rows from the back).
struct XRow {
    int x, meta, beg, len;
    double c0, c1, c2;
    uint32_t mk;
    int pad;
};
constexpr int kXcap = 16384;  // deferred long rows per worker (beyond: walked in-lane)

struct Scratch {
    uint32_t *mark;            // epoch<<2 | state
    unsigned long long *lowrec;  // (epoch << 32) | old d, written by the lowering thread
    double *dacc;              // Delta-delta accumulator; all-zero between jobs
    int32_t *Dv;               // down set D in BFS level order (also the static BFS order)
    int32_t *Dold;             // old d of D[i]
    double *Dsig;              // old sigma of D[i]
    int32_t *Doff;             // level offsets of D (also static level offsets), n+2
    int32_t *U0, *U1;          // up frontier overflow ping-pong
    int32_t *Rv, *Rl;          // removal-push targets and their levels (Case 3)
    int32_t *Bq;               // long-row queue of the current level, n per worker
    struct XRow *X;            // wide up levels: long rows beyond one chunk, kXcap per worker
    int32_t *Wul, *Wlev;       // window of insertions: u_low and seed level, wcap per worker
    int32_t wcap;              // window capacity (insertions per job)
    uint32_t *wepoch;          // per-worker epoch counter
};

// ---------------------------------------------------------------------------
// Loads: the immutable graph through the read-only path; mutable state with
// plain (L1-cacheable) loads.  A worker CTA is the only writer of its root's
// records and of its scratch during a launch; every cross-thread dependency is
// ordered by __syncthreads() (which makes all earlier global writes and
// atomics of the block visible to it); the same-level races the algorithm
// tolerates (lowering, claims) are resolved by atomics, so a stale line can
// only cost a redundant atomic, never a wrong value.  L1 is invalidated
// between launches.
__device__ __forceinline__ int ldg_i(const int32_t *p) { return __ldg(p); }


// Adjacency row of v, restricted to batch entries with insertion index <= limit
// (canonical order: base row, then inserted neighbours in insertion order).
__device__ __forceinline__ int2 row_of(const GView &g, int v, int limit) {
    int rb = ldg_i(g.rp + v);
    int re = ldg_i(g.rp + v + 1) & kMask;
    if (rb < 0) {
        rb &= kMask;
        int2 xi = __ldg(g.xinfo + v);
        int vis = 0;
        while (vis < xi.y && ldg_i(g.xtag + xi.x + vis) <= limit) ++vis;
        re -= xi.y - vis;
    }
    return make_int2(rb, re);
}

// Does the sorted range scol[lo, hi) hold p?  A 16-ary search: every step
// issues 16 independent probes (one memory round trip) and keeps the 1/16 of
// the range that can hold p, so a row of 10^4 entries takes 4 dependent round
// trips instead of a binary search's 14.
__device__ __forceinline__ bool sorted_range_contains(const int32_t *scol, int lo, int hi, int p) {
    constexpr int K = 16;
    while (hi - lo > K) {
        const int step = (hi - lo + K - 1) / K;
        int q[K];
#pragma unroll
        for (int k = 0; k < K; ++k) q[k] = lo + k * step < hi ? ldg_i(scol + lo + k * step) : INT32_MAX;
        int c = 0;
#pragma unroll
        for (int k = 0; k < K; ++k) c += q[k] <= p ? 1 : 0;
        if (c == 0) return false;  // p is below the range
        lo += (c - 1) * step;       // scol[lo] <= p < the next probe
        hi = min(hi, lo + step);
    }
    int q[K];
#pragma unroll
    for (int k = 0; k < K; ++k) q[k] = lo + k < hi ? ldg_i(scol + lo + k) : -1;
    bool f = false;
#pragma unroll
    for (int k = 0; k < K; ++k) f |= q[k] == p;
    return f;
}

// Is p a neighbour of x in the graph as of insertion `limit`?  A search of x's
// sorted row (all entries), then a batch-entry visibility check.
__device__ __forceinline__ bool adjacent_visible(const GView &g, int x, int p, int limit) {
    const int rb = ldg_i(g.rp + x);
    if (!sorted_range_contains(g.scol, rb & kMask, ldg_i(g.rp + x + 1) & kMask, p)) return false;
    if (rb < 0) {  // x has entries of the current batch: is (x, p) one of them, and visible?
        const int2 xi = __ldg(g.xinfo + x);
        for (int k = 0; k < xi.y; ++k)
            if (ldg_i(g.xnbr + xi.x + k) == p) return ldg_i(g.xtag + xi.x + k) <= limit;
    }
    return true;
}

// Is (x, p) an edge inserted by insertion g0 .. lim of the current batch?  x
// must have batch entries (rp[x] flagged).  A job's pushes subtract the old
// contribution sigma[p]/sigma_old(x)*(1+delta_old(x)) only over edges that
// existed before the job -- for a single insertion this is Alg. 2's guard
// "v != u_high or w != u_low", for a Case-2 group every edge of it.
__device__ __forceinline__ bool new_edge(const GView &g, int x, int p, int g0, int lim) {
    const int2 xi = __ldg(g.xinfo + x);
    for (int k = 0; k < xi.y; ++k)
        if (ldg_i(g.xnbr + xi.x + k) == p) {
            const int t = ldg_i(g.xtag + xi.x + k);
            return t >= g0 && t <= lim;
        }
    return false;
}

// ---------------------------------------------------------------------------
// Level processing (the paper's node-based parallelism, Sec. III, P:272-274,
// re-mapped for B200): the vertices of one BFS level are split by row length.
//  * short rows (<= kSmallDeg entries): one lane walks the whole row in
//    canonical order with kRowUnroll entries in flight (bit-exact pull sums);
//  * long rows (hubs): processed by the whole CTA with their entries
//    flattened (every thread takes a few entries per step, gathers hoisted),
//    per-row reductions through warp-aggregated shared-memory fp64 atomics --
//    the load-balanced "advance" of Merrill et al. [19] (cited at P:322).

// Sequential walk of one (small) row in canonical order: columns, then the
// neighbours' distances, then -- only for entries passing want(d) -- their
// (sigma, delta) pair and mk[y] (if mk), kRowUnroll entries in flight; then
// f(y, d, sd, mark) runs in order.
#ifndef DBC_ROW_UNROLL
// 64-register builds (>= 1024 resident threads per CTA launch bound) keep 4
// entries in flight per lane: 8 would spill the gathered arrays
#define DBC_ROW_UNROLL ((DBC_BLOCK * DBC_MINB >= 1024) ? 4 : 8)
#endif
constexpr int kRowUnroll = DBC_ROW_UNROLL;
template <class Want, class F>
__device__ __forceinline__ void row_walk(const GView &g, const Root &st, const uint32_t *mk,
                                         int2 r, Want want, F f) {
    for (int j = r.x; j < r.y; j += kRowUnroll) {
        int y[kRowUnroll], dy[kRowUnroll];
        double2 q[kRowUnroll];
        uint32_t mm[kRowUnroll];
#pragma unroll
        for (int u = 0; u < kRowUnroll; ++u) y[u] = (j + u < r.y) ? ldg_i(g.col + j + u) : -1;
#pragma unroll
        for (int u = 0; u < kRowUnroll; ++u) dy[u] = (y[u] >= 0) ? st.dist(y[u]) : kInf;
#pragma unroll
        for (int u = 0; u < kRowUnroll; ++u) {
            const bool w = y[u] >= 0 && want(dy[u]);
            q[u] = w ? st.sd[y[u]] : make_double2(0.0, 0.0);
            mm[u] = (mk && w) ? mk[y[u]] : 0u;
        }
#pragma unroll
        for (int u = 0; u < kRowUnroll; ++u)
            if (y[u] >= 0) f(y[u], dy[u], q[u], mm[u]);
    }
}

// --- long rows: rounds of up to kBig rows staged in shared memory -----------
constexpr int kBig = 128;     // long rows per round (down phase / static)
constexpr int kUnroll = 4;    // entries per thread in flight

struct BigSmem {
    int idx[kBig];    // item index (caller's list) of each long row
    int v[kBig];      // vertex
    int b[kBig];      // row begin
    int off[kBig + 1];  // exclusive scan of row lengths; off[m] = total
    double acc[kBig];   // per-row reduction
    double c0[kBig];    // per-row constant of the caller
    unsigned mk[kBig];  // per-row level-2 predecessor mask being built
    int ext[kBig];      // per-row: a predecessor outside D was seen (update down phase)
    int m;            // rows in this round
};

// Pass over `count` items: short rows processed inline by their lane, long
// rows handed (as item indices) to enqueue().
template <class Get, class Small, class Enq>
__device__ __forceinline__ void split_pass(int count, const GView &g, int limit, Get get,
                                           Small small, Enq enqueue) {
    for (int idx = threadIdx.x; idx < count; idx += kBlock) {
        int v = 0;
        if (!get(idx, v)) continue;
        const int2 r = row_of(g, v, limit);
        if (r.y - r.x > kSmallDeg)
            enqueue(idx);
        else
            small(idx, v, r);
    }
}

// Load a round of m <= kBig queued long rows (rows, offsets).  Caller must
// __syncthreads() before (queue complete); ends with a barrier.
template <class Fetch, class GetV>
__device__ __forceinline__ void big_load(BigSmem &S, int m, Fetch fetch, GetV getv,
                                         const GView &g, int limit) {
    const int tid = threadIdx.x;
    if (tid < m) {
        const int idx = fetch(tid);
        const int v = getv(idx);
        const int2 r = row_of(g, v, limit);
        S.idx[tid] = idx;
        S.v[tid] = v;
        S.b[tid] = r.x;
        S.off[tid + 1] = r.y - r.x;
        S.acc[tid] = 0.0;
    }
    if (tid == 0) {
        S.off[0] = 0;
        S.m = m;
    }
    __syncthreads();
    if (tid < 32) {  // inclusive scan of off[1..m] by warp 0 (m <= kBig = 4*32)
        int vals[kBig / 32];
        int run = 0;
#pragma unroll
        for (int q = 0; q < kBig / 32; ++q) {
            const int i = tid * (kBig / 32) + q;
            vals[q] = (i < m) ? S.off[i + 1] : 0;
            run += vals[q];
        }
        int incl = run;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(kFull, incl, o);
            if (tid >= o) incl += y;
        }
        int ex = incl - run;
#pragma unroll
        for (int q = 0; q < kBig / 32; ++q) {
            const int i = tid * (kBig / 32) + q;
            ex += vals[q];
            if (i < m) S.off[i + 1] = ex;
        }
    }
    __syncthreads();
}

// warp-aggregated shared-memory accumulation of c into acc[t] (all lanes call;
// t < 0 = no contribution)
__device__ __forceinline__ void acc_add(double *acc, int t, double c) {
    const int lane = threadIdx.x & 31;
    const int t0 = __shfl_sync(kFull, t, 0);
    const bool uni = __all_sync(kFull, t == t0 || t < 0);
    if (uni) {
        if (t0 >= 0) {
#pragma unroll
            for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(kFull, c, o);
            if (lane == 0 && c != 0.0) atomicAdd(acc + t0, c);
        }
    } else if (t >= 0 && c != 0.0) {
        atomicAdd(acc + t, c);
    }
}

// Flattened pass over all entries of a loaded round (strided mapping).
// f(t, y, d, sd) returns a contribution summed into S.acc[t]; sd is gathered
// only for entries passing want(d).  Ends with a barrier.
template <class Want, class F>
__device__ __forceinline__ void big_entries(BigSmem &S, const GView &g, const Root &st, Want want, F f) {
    const int tid = threadIdx.x;
    const int m = S.m, E = S.off[m];
    for (int base = 0; base < E; base += kUnroll * kBlock) {
        int t[kUnroll], y[kUnroll], dy[kUnroll];
        double2 q[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
            const int e = base + u * kBlock + tid;
            t[u] = -1;
            y[u] = 0;
            if (e < E) {
                int lo = 0, hi = m - 1;  // last t with off[t] <= e
                while (lo < hi) {
                    const int mid = (lo + hi + 1) >> 1;
                    if (S.off[mid] <= e) lo = mid; else hi = mid - 1;
                }
                t[u] = lo;
                y[u] = ldg_i(g.col + S.b[lo] + (e - S.off[lo]));
            }
        }
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) dy[u] = (t[u] >= 0) ? st.dist(y[u]) : kInf;
#pragma unroll
        for (int u = 0; u < kUnroll; ++u)
            q[u] = (t[u] >= 0 && want(dy[u])) ? st.sd[y[u]] : make_double2(0.0, 0.0);
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
            double c = 0.0;
            if (t[u] >= 0) c = f(t[u], y[u], dy[u], q[u]);
            acc_add(S.acc, t[u], c);
        }
    }
    __syncthreads();
}

// --- up phase: chunked flattened level pass ----------------------------------
constexpr int kChunk = 512;   // items per chunk (shared memory; one layout for every CTA width,
                              // so owners and helpers of different widths share the help board)
constexpr int kUcap = 1024;   // up-frontier entries kept in shared memory
constexpr int kMetaUp = 1, kMetaNotPulled = 2, kMetaMask = 4;
constexpr int kMetaNew = 8;  // down row with batch entries: its pushes check new_edge()
constexpr int kMetaExt = 16; // down row with a predecessor outside D: it has pushes to make
#ifndef DBC_FLAT_U
#define DBC_FLAT_U 4
#endif
constexpr int kFlatU = DBC_FLAT_U;  // contiguous entries per thread per step
constexpr int kWindow = 16384;  // default insertions per Mode-A job (DBC_WINDOW overrides)
constexpr int kAdjCap = 256;  // longest root row kept in shared memory (level-2 shortcut)

struct ChunkSmem {
    int v[kChunk];
    int meta[kChunk];
    int beg[kChunk];
    int off[kChunk + 1];
    double acc[kChunk], c0[kChunk], c1[kChunk], c2[kChunk];
    unsigned mk[kChunk];  // level-2 predecessor mask of masked up items
};

// exclusive scan in place of off[1..cnt] (lengths) -> off[0..cnt]; ends with a barrier
__device__ __forceinline__ void chunk_scan(int *off, int cnt) {
    __shared__ int ws[kWarps];
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    constexpr int per = kChunk >= kBlock ? kChunk / kBlock : 1;  // items per thread
    int vals[per];
    int run = 0;
#pragma unroll
    for (int q = 0; q < per; ++q) {
        const int i = tid * per + q;
        vals[q] = (i < cnt) ? off[i + 1] : 0;
        run += vals[q];
    }
    int incl = run;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(kFull, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) ws[wid] = incl;
    __syncthreads();
    int wbase = 0;
    for (int w = 0; w < wid; ++w) wbase += ws[w];
    int ex = wbase + incl - run;
#pragma unroll
    for (int q = 0; q < per; ++q) {
        const int i = tid * per + q;
        ex += vals[q];
        if (i < cnt) off[i + 1] = ex;
    }
    if (tid == 0) off[0] = 0;
    __syncthreads();
}

// Flattened entries [0, E) of the chunk's rows (off = exclusive offsets of cnt
// rows): thread tid takes kFlatU consecutive entries per step (one binary
// search, then linear advance), gathers columns and record halves up front and
// calls f(t, y, d, sd, mark) (sd, mark gathered for want(d)); if acc != nullptr
// the returned contribution is
// summed into acc[t].  Ends with a barrier.
// kSd = false: sd is not gathered (f sees zeros), only mark.
template <bool kCG = false, bool kSd = true, class Want, class Col, class F>
__device__ __forceinline__ void flat_entries(const int *off, int cnt, int E, Col colf, const Root &st,
                                             const uint32_t *mk, Want want, double *acc, F f, int Ebeg = 0) {
    const int tid = threadIdx.x;
    for (int base = Ebeg; base < E; base += kBlock * kFlatU) {
        const int e0 = base + tid * kFlatU;
        int t[kFlatU], y[kFlatU], dy[kFlatU];
        double2 q[kFlatU];
        uint32_t mm[kFlatU];
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
        for (int u = 0; u < kFlatU; ++u) {
            const bool w = t[u] >= 0 && want(dy[u]);
            q[u] = (kSd && w) ? (kCG ? __ldcg(st.sd + y[u]) : st.sd[y[u]]) : make_double2(0.0, 0.0);
            mm[u] = (mk && w) ? (kCG ? __ldcg(mk + y[u]) : mk[y[u]]) : 0u;
        }
#pragma unroll
        for (int u = 0; u < kFlatU; ++u) {
            double c = 0.0;
            if (t[u] >= 0) c = f(t[u], y[u], dy[u], q[u], mm[u]);
            if (acc) acc_add(acc, t[u], c);
        }
    }
    __syncthreads();
}

// ---------------------------------------------------------------------------
// Level-2 predecessor masks (roots with at most kMaskDeg neighbours): bit j of
// mask[x] is set iff x (a level-2 vertex) is adjacent to the j-th neighbour of
// the root in the root's canonical row.  The level-1 predecessors of a level-2
// vertex -- the pushes of the up phase into level 1 -- then come from one
// gather instead of a scan of x's row.  Valid for vertices with d == 2 only.
constexpr int kMaskDeg = 32;

// (Re)build all masks of one root from its row rs (as of `limit`): clear the
// masks of every level-2 vertex, then OR in one bit per level-1 neighbour.
// Whole CTA; ends with a barrier.
__device__ __forceinline__ void build_l2masks(const GView &g, const Root &st, uint32_t *mask,
                                              int2 rs, int limit) {
    const int ds = rs.y - rs.x;
    for (int pass = 0; pass < 2; ++pass) {
        for (int j = 0; j < ds; ++j) {
            const int p = ldg_i(g.col + rs.x + j);
            const int2 rp = row_of(g, p, limit);
            for (int e = rp.x + (int)threadIdx.x; e < rp.y; e += kBlock) {
                const int x = ldg_i(g.col + e);
                if (st.dist(x) != 2) continue;
                if (pass == 0)
                    mask[x] = 0u;
                else
                    atomicOr(mask + x, 1u << j);
            }
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------
// Cooperative help: a worker whose up-level push pass (C2)
// has many entries publishes it on a help board; workers that have run out of
// roots join it block by block.  Per owner: a packed word
//   bit 63 open | bits 40..59 blocks | bits 16..35 next block | bits 0..15 seq
// (helpers grab a block with one atomicAdd of 1 << 16), a done counter, the
// job context, a global mirror of the chunk and a global append list.
// flattened passes (C1 pull, C2 push) are published when they have at least
// UpdateArgs.he_min blocks of he_entries entries (defaults 3 x 4096)
struct HelpCtx {
    int root_slot, l, g0, lim, cnt, nblocks, E2;  // g0..lim: the job's insertions
    uint32_t E;  // epoch << 2 of the job
    int kind;    // 0: C2 push pass of a published chunk; 1: a down-phase level;
                 // 2: C1 delta-pull pass of a chunk; 3: the Case-3 removal pass over D;
                 // 4: the long rows of a down level, entry-balanced (E2 entries, cnt rows);
                 // 5: the in-lane item pass of a wide up level (cnt items, E2 = |down segment|)
    int lb;      // kind 1: the level's first position in D; kind 5: b0
    int mvalid;  // kind 1: level-2 masks are maintained
    int aux;     // kind 5: |up frontier| | (its overflow list is U1) << 30
};
struct HelpBoard {
    unsigned long long *word;  // [workers]
    int *done;                 // [workers]
    HelpCtx *ctx;              // [workers]
    ChunkSmem *mir;            // [workers]
    int *gapp;                 // [workers] global append counters
    int32_t *gU;               // [workers][n] global append lists
    int *roots_left;           // [0] root chains not yet finished (both lanes), [1] open wide requests,
                               // [2] idle workers, [3..5] = {k_loc, 0, 0}: the per-batch reset source
    int *low;                  // [workers] kind 1: a distance was lowered in the helped level;
                               // kind 3: deepest removal-target level
    int nworkers;
    int *gbig;                 // [workers][2] kind 1: long rows queued in the owner's Bq, their entries
};
__device__ __forceinline__ unsigned long long help_pack(int open, int nblocks, int next, int seq) {
    return ((unsigned long long)(open ? 1 : 0) << 63) | ((unsigned long long)(nblocks & 0xFFFFF) << 40) |
           ((unsigned long long)(next & 0xFFFFF) << 16) | (unsigned long long)(seq & 0xFFFF);
}
__device__ __forceinline__ bool help_open(unsigned long long w) { return (w >> 63) != 0; }
__device__ __forceinline__ int help_nblocks(unsigned long long w) { return (int)((w >> 40) & 0xFFFFF); }
__device__ __forceinline__ int help_next(unsigned long long w) { return (int)((w >> 16) & 0xFFFFF); }
__device__ __forceinline__ int help_seq(unsigned long long w) { return (int)(w & 0xFFFF); }

// ---------------------------------------------------------------------------
// kernel entry points (defined in static_brandes.cu / update.cu)
struct UpdateArgs {
    GView g;
    int32_t n;
    int32_t k_loc;
    const int32_t *roots;  // local roots (internal ids), [k_loc]
    int32_t *d;            // [k_loc][n]
    double2 *sd;           // [k_loc][n]
    double *bc;
    const int32_t *ins_u, *ins_v;  // batch, device (internal ids)
    int32_t ins_begin, ins_end;    // batch-local insertion range of this launch
    Scratch ws;
    int32_t *next_slot;            // work counter (zeroed before launch)
    unsigned long long *stats;     // kStCount counters
    int32_t *err;
    uint32_t *l2mask;              // [k_loc][n] level-2 predecessor masks (see below)
    int32_t *mask_ds;              // [k_loc] root degree the masks were built for (-1: none)
    unsigned long long *root_prof; // nullable: per local slot {t_begin, t_end, jobs, ...}
    const int32_t *slot_list;      // nullable: the slots this launch processes (else 0..k_loc-1)
    int32_t slot_count;            // entries of slot_list
    int32_t worker_base;           // scratch index of CTA 0
    const int32_t *steal_list;     // nullable: the other lane's slots, taken once this list is done
    int32_t steal_count;
    int32_t *steal_next;           // the other lane's counter
    HelpBoard help;                // help.word == nullptr: no cooperative help
    int32_t merge;                 // 1: a window of ws.wcap insertions per job; 0: one per insertion
    long long *scen;               // nullable: scenario log [batch insertion][k_loc] (merge == 0)
    int32_t del;                   // 1: ins_u/ins_v[ins_begin] is an edge DELETION (already tombstoned)
    int32_t lowdeg;                // 1: rows are short: up levels of any size are walked in-lane
    int32_t hd_min, hd_block;      // down levels of >= hd_min items are published in hd_block blocks
    int32_t he_entries, he_min;    // flattened passes: entries per help block, minimum blocks
    int32_t busy_help;             // blocks a busy worker takes per poll of the board (0: only idle workers help)
    int32_t busy_min;              // busy workers take blocks of passes of at least this many blocks
    int32_t dl_min;                // down levels whose long rows hold >= dl_min entries: entry-balanced pass
    int32_t wide_inlane;           // up levels of <= wide_inlane items per thread: short rows in-lane, long rows chunked
    int32_t trace_slot;            // -DDBC_PHASE_TIMERS builds: time this slot only (-1: all)
    int32_t static_slots;          // unused (kept zero)
    void *lean_board;              // update_lean.cu help board (nullptr: no cooperative help)
    int32_t pull_delta;            // update_lean.cu: DBC_FLAG_PULL_DELTA (every touched vertex pulls delta)
    int32_t short_mult;            // update_lean.cu: level-2 up rows longer than short_mult x deg(root)
                                   // find their predecessors by probing adj(root)
};

struct StaticArgs {
    int32_t exact_delta;  // DBC_FLAG_PULL_DELTA: long rows' delta re-summed in canonical order
    GView g;
    int32_t n;
    int32_t k_loc;
    const int32_t *roots;
    int32_t *d;
    double2 *sd;
    double *bc;
    Scratch ws;
    int32_t *next_slot;
    unsigned long long *stats;
    int32_t *err;
    uint32_t *l2mask;
    int32_t *mask_ds;
};

// Edge-based parallel update (edge_parallel.cu, DBC_FLAG_EDGE_PARALLEL).
struct EdgeArgs {
    GView g;
    int32_t n;
    int32_t k_loc;
    const int32_t *roots;
    int32_t *d;
    double2 *sd;
    double *bc;
    const int32_t *ins_u, *ins_v;
    int32_t ins;                // the insertion of this launch (batch-local)
    Scratch ws;
    double *odel;               // [workers][n] old delta by vertex
    const int32_t *src, *tag;   // [nnz] entry source / insertion index (-1: base)
    int32_t nnz;
    int32_t *next_slot;
    unsigned long long *stats;
    int32_t *err;
};
int launch_edge_coo(const GView &g, int32_t n, int32_t *src, int32_t *tag, cudaStream_t s);
void launch_edge_update(const EdgeArgs &a, int workers, cudaStream_t s);

void launch_update_256(const UpdateArgs &a, int workers, cudaStream_t s);
// update_lean.cu, one job per insertion: 128-, 256-, 512- and 1024-thread builds
void launch_update_lean_128(const UpdateArgs &a, int workers, cudaStream_t s);
void launch_update_lean_256(const UpdateArgs &a, int workers, cudaStream_t s);
void launch_update_lean_512(const UpdateArgs &a, int workers, cudaStream_t s);
void launch_update_lean_512x2(const UpdateArgs &a, int workers, cudaStream_t s);  // 64 registers, two per SM
void launch_update_lean_1024(const UpdateArgs &a, int workers, cudaStream_t s);
int lean_resident_128();  // resident CTAs per SM of each build
int lean_resident_256();
int lean_resident_512();
int lean_resident_512x2();
int lean_resident_1024();
size_t lean_board_bytes();
void launch_update_512x2(const UpdateArgs &a, int workers, cudaStream_t s);  // 64 regs, 2 CTAs/SM
void launch_update_1024(const UpdateArgs &a, int workers, cudaStream_t s);   // heavy lane, 64 regs
void launch_update_128(const UpdateArgs &a, int workers, cudaStream_t s);
void launch_update_512(const UpdateArgs &a, int workers, cudaStream_t s);
void launch_static_256(const StaticArgs &a, int workers, cudaStream_t s);
void launch_static_128(const StaticArgs &a, int workers, cudaStream_t s);
void launch_static_512(const StaticArgs &a, int workers, cudaStream_t s);   // 64 regs, 2 CTAs/SM
void launch_static_1024(const StaticArgs &a, int workers, cudaStream_t s);  // 64 regs, 1 CTA/SM

// Multi-source static Brandes (msbrandes.cu): one wave of 32-root groups.
struct MsArgs {
    GView g;
    int32_t n;
    int32_t k_loc;
    const int32_t *roots;
    int32_t g0, ng;        // groups g0 .. g0 + ng - 1 (slots 32 R g .. 32 R g + 32 R - 1)
    double *sg;            // [ng][n][32 R] sigma (zeroed)
    double *q;             // [ng][n][32 R] q = (1 + delta) / sigma (zeroed)
    uint8_t *lv;           // [ng][n][32 R] BFS level, 255 = unreached (0xff-filled)
    // masks over the 32 R roots of a group (R = 1: uint32, R = 2: uint64)
    void *vis;             // [ng][n] roots that reached the vertex (zeroed)
    void *nm;              // [ng][3][n] level masks, level j in array j % 3 (zeroed)
    int32_t *vq;           // [ng][vcap] level lists (vertex)
    void *vm;              // [ng][vcap] ... and its roots at that level
    int2 *tq;              // [ng][tcap] row-chunk tasks {vq index, chunk}
    int32_t *toff;         // [ng][max levels + 3] first task of each level
    int32_t *ctr;          // [ng] {vcount, tcount, overflow, pad} (zeroed)
    unsigned *bar;         // grid barrier {count, generation} (zeroed)
    int64_t vcap, tcap;
    int32_t chunk;         // row entries per task
    int32_t *d;            // root-major state (written for the wave's slots)
    double2 *sd;
    double *bc;
    unsigned long long *stats;
    int32_t *err;
};
int ms_static_max_groups();
int ms_static_max_levels();
size_t ms_static_counter_bytes(int ng);
int ms_static_resident(int nsm, int r);  // r = roots per lane (1 or 2)
cudaError_t launch_static_ms(const MsArgs &a, int r, int grid, cudaStream_t s);
void launch_static_l2mask(const StaticArgs &a, cudaStream_t s);

}  // namespace dbc
