// dbc_internal.cuh -- shared device-side definitions of libdbc (B200 / sm_100a).
//
// Layout in HBM:
//   graph   rp int32[n+1] (bit 31 of rp[v] = "row v has entries of the current
//           batch"), col int32[cap]; for flagged rows xinfo[v] = {first tag
//           index, count} and xtag[] = batch-local insertion index of each batch
//           entry, in row order.  Row v = col[rp[v] .. rp[v+1]) (masked): the
//           base part, then the current batch's entries sorted by insertion index.
//   state   d int32[k_loc][n], sd double2[k_loc][n] = (sigma, delta) per vertex,
//           root-major (each root's arrays contiguous), bc double[n].
//   scratch per persistent worker CTA, n-sized arrays (epoch-tagged, never
//           cleared between jobs -- no O(n) work per root per insertion,
//           SURVEY.md Sec. 7 hard part (iii)).
#pragma once

#include <cstdint>
#include <type_traits>

#include <cuda_runtime.h>

namespace dbc {

constexpr int kBlock = 256;              // threads per worker CTA
constexpr int kWarps = kBlock / 32;
constexpr int kSmallDeg = 32;            // rows <= this are walked by one lane
constexpr uint32_t kFull = 0xffffffffu;
constexpr int32_t kInf = INT32_MAX;
constexpr int32_t kMask = 0x7fffffff;
constexpr uint32_t kDown = 1u;           // mark state: in the down set D (Alg. 2 t[v] = down)
constexpr uint32_t kUp = 2u;             // mark state: found by the up phase (t[v] = up)
constexpr double kExact = 9007199254740992.0;  // 2^53

enum ErrBits : int { kErrNumeric = 1, kErrOverflow = 2 };

// Counters accumulated by the kernels (device, u64).
enum StatIdx : int {
    kStCase1 = 0, kStCase2, kStCase3, kStTouched, kStDown, kStScanned, kStBytes,
    kStStaticBytes, kStCount
};

struct GView {
    const int32_t *__restrict__ rp;
    const int32_t *__restrict__ col;
    const int2 *__restrict__ xinfo;
    const int32_t *__restrict__ xtag;
};

// Scratch of the persistent workers (one CTA = one worker), each array
// worker-major with stride n.
struct Scratch {
    uint32_t *mark;            // epoch<<2 | state
    unsigned long long *lowrec;  // (epoch << 32) | old d, written by the lowering thread
    double *dacc;              // Delta-delta accumulator; all-zero between jobs
    int32_t *Dv;               // down set D in BFS level order (also the static BFS order)
    int32_t *Dold;             // old d of D[i]
    double *Dsig;              // old sigma of D[i]
    int32_t *Doff;             // level offsets of D (also static level offsets), n+2
    int32_t *U0, *U1;          // up frontier ping-pong
    int32_t *Rv, *Rl;          // removal-push targets and their levels (Case 3)
    uint32_t *wepoch;          // per-worker epoch counter
};

// ---------------------------------------------------------------------------
// loads: immutable graph via the read-only path, mutable state via L2 (.cg) so
// values written by atomics of the same kernel are never served stale from L1.
__device__ __forceinline__ int ldg_i(const int32_t *p) { return __ldg(p); }
__device__ __forceinline__ int ldcg_i(const int32_t *p) { return __ldcg(p); }
__device__ __forceinline__ double ldcg_d(const double *p) { return __ldcg(p); }
__device__ __forceinline__ double2 ldcg_d2(const double2 *p) { return __ldcg(p); }
__device__ __forceinline__ uint32_t ldcg_u(const uint32_t *p) { return __ldcg(p); }
__device__ __forceinline__ unsigned long long ldcg_ull(const unsigned long long *p) { return __ldcg(p); }

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

template <int G>
__device__ __forceinline__ double group_sum(double x) {
    if constexpr (G == 32) {
#pragma unroll
        for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(kFull, x, o);
    }
    return x;  // butterfly: every lane ends with the same (commutative) value
}

template <int G>
__device__ __forceinline__ void group_sync() {
    if constexpr (G == 32) __syncwarp();
}

using G1 = std::integral_constant<int, 1>;
using G32 = std::integral_constant<int, 32>;

// Two-tier node-parallel mapping of a vertex list onto a CTA (the paper's
// node-based parallelism, Sec. III, re-mapped for 32-wide warps):
// each warp takes 32 consecutive items, one per lane; rows of <= kSmallDeg
// entries are walked sequentially by their lane (canonical order for free),
// longer rows are walked by the whole warp, one row at a time.
//   get(idx, &v) -> bool   : item idx is active, vertex v
//   need_row(idx, v) -> bool: whether the body needs the adjacency row
//   body(G, idx, v, row, gl): gl = lane within the group (0 for G1)
template <class Get, class NeedRow, class Body>
__device__ __forceinline__ void two_tier(int count, const GView &g, int limit, Get get,
                                         NeedRow need_row, Body body) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int base = warp * 32; base < count; base += kWarps * 32) {
        const int idx = base + lane;
        int v = 0;
        bool valid = idx < count && get(idx, v);
        int2 r = make_int2(0, 0);
        if (valid && need_row(idx, v)) r = row_of(g, v, limit);
        const bool big = valid && (r.y - r.x) > kSmallDeg;
        if (valid && !big) body(G1{}, idx, v, r, 0);
        unsigned bm = __ballot_sync(kFull, big);
        while (bm) {
            const int src = __ffs(bm) - 1;
            bm &= bm - 1;
            const int bidx = __shfl_sync(kFull, idx, src);
            const int bv = __shfl_sync(kFull, v, src);
            int2 br;
            br.x = __shfl_sync(kFull, r.x, src);
            br.y = __shfl_sync(kFull, r.y, src);
            body(G32{}, bidx, bv, br, lane);
        }
    }
}

// ---------------------------------------------------------------------------
// kernel entry points (defined in graph.cu / static_brandes.cu / update.cu)
struct UpdateArgs {
    GView g;
    int32_t n;
    int32_t k_loc;
    const int32_t *roots;  // local roots, [k_loc]
    int32_t *d;
    double2 *sd;
    double *bc;
    const int32_t *ins_u, *ins_v;  // batch, device
    int32_t ins_begin, ins_end;    // batch-local insertion range of this launch
    Scratch ws;
    int32_t *next_slot;            // work counter (zeroed before launch)
    unsigned long long *stats;     // kStCount counters
    int32_t *err;
};

struct StaticArgs {
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
};

void launch_update(const UpdateArgs &a, int workers, cudaStream_t s);
void launch_static(const StaticArgs &a, int workers, cudaStream_t s);

}  // namespace dbc
