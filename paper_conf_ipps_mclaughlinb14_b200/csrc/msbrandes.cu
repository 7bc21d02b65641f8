// msbrandes.cu -- K1 for low-diameter graphs: multi-source static Brandes,
// 32 roots per warp (one root per lane).  Same state as static_brandes.cu
// (Alg. 1; Eqs. (2)-(3)): d and sigma bit-exact
// (sigma summed left to right in canonical row order; a row split over several
// tasks adds its chunk partials atomically -- integer-valued sums, exact in any
// order below 2^53, re-summed in canonical order at or above it), delta and BC
// within the north star's tolerances (Eq. (2) regrouped, below).
//
// B200 design (DESIGN.md Sec. 6 K1-MS).  The per-root kernel gathers a 4-byte
// distance and an 8-byte sigma per (root, neighbour) -- a 32-byte sector each.
// Here a group of 32 roots is traversed together: per vertex a 32-bit lane mask
// per BFS level (nm) and sigma held vertex-major (double[n][32]) in scratch, so
// one neighbour gather serves the 32 roots (one sector of masks, then the sigma
// line of the lanes whose bit is set), and a vertex's row is scanned once per
// distinct level it has among the 32 roots (a handful on low-diameter graphs),
// not once per root.  A persistent cooperative grid runs all groups of a wave
// in lockstep levels separated by grid barriers:
//   pass A (level L): expand -- lanes over the entries of the frontier rows; a
//          neighbour w gets the lanes m(u) & ~vis(w) by atomicOr into the
//          level-(L+1) mask; the first claimer appends w to level L+1;
//   pass B (level L+1): sigma pull -- lane = root, each row's predecessors at
//          level L summed in canonical order;
//   backward (level L = max .. 1): delta by Eq. (2) regrouped as
//          delta(w) = sigma(w) * sum_y q(y), q(y) = (1 + delta(y)) / sigma(y),
//          stored once a vertex's delta is final -- one gather per successor
//          instead of two and a division;
//   final:  tiles transposed into the root-major state of the dynamic kernels.
// Work unit: a task = a row chunk of <= `chunk` entries of one (vertex, level);
// a warp takes 32 consecutive tasks (their metadata in one round of loads,
// one task per lane) and walks their entries flattened, 32 per step.
// BC gets one atomic add per (vertex, level, group).  A group whose BFS passes level kMsMaxLev or whose
// level lists outgrow their capacity sets an overflow flag and the host
// recomputes with the per-root kernel; so does DBC_FLAG_PULL_DELTA (bitwise
// delta needs Eq. (2)'s own order).
#include "dbc_internal.cuh"

namespace dbc {

namespace {

constexpr int kMsThreads = 256;
constexpr int kMsMaxG = 64;      // groups per wave (lockstep)
constexpr int kMsMaxLev = 254;   // deeper BFS: the per-root kernel
constexpr int kMsUnroll = 8;     // contributing entries whose gathers are in flight together

// R roots per lane (a group of 32 R roots): lane l holds roots l + 32 j, j < R;
// a vertex's lanes at a level form one R * 32-bit mask.
template <int R> struct MaskOf;
template <> struct MaskOf<1> { using T = uint32_t; };
template <> struct MaskOf<2> { using T = unsigned long long; };
__device__ __forceinline__ int popc_m(uint32_t x) { return __popc(x); }
__device__ __forceinline__ int popc_m(unsigned long long x) { return __popcll(x); }
template <class Mk> __device__ __forceinline__ bool bit(Mk m, int b) { return (m >> b) & 1u; }

struct MsGroup {  // per-group counters (device)
    int vcount, tcount, overflow, pad;
};

__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// Grid-wide barrier of a cooperative launch (all CTAs co-resident).
__device__ __forceinline__ void grid_sync(unsigned *bar) {
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned gen = ld_acquire(bar + 1);
        __threadfence();
        if (atomicAdd(bar, 1u) == gridDim.x - 1) {
            atomicExch(bar, 0u);
            __threadfence();
            atomicAdd(bar + 1, 1u);
        } else {
            while (ld_acquire(bar + 1) == gen) __nanosleep(32);
        }
        __threadfence();
    }
    __syncthreads();
}

// Phase clock (block 0, thread 0, after a grid barrier; dbc_debug_counters):
// stats[kStTrace0 + 2 i] = kind << 16 | level, + 1 = %globaltimer (ns).
__device__ __forceinline__ void ms_trace(unsigned long long *stats, int kind, int level) {
    if (blockIdx.x != 0 || threadIdx.x != 0) return;
    const unsigned long long i = stats[kStTraceN];
    if (i >= kTraceCap) return;
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    stats[kStTrace0 + 2 * i] = ((unsigned long long)kind << 16) | (unsigned)level;
    stats[kStTrace0 + 2 * i + 1] = t;
    stats[kStTraceN] = i + 1;
}

__device__ __forceinline__ int2 full_row(const GView &g, int v) {
    return make_int2(ldg_i(g.rp + v) & kMask, ldg_i(g.rp + v + 1) & kMask);
}

template <int R>
struct Ms {
    using Mk = typename MaskOf<R>::T;
    static constexpr int G = 32 * R;  // roots per group
    const MsArgs &a;
    size_t n;
    int lane, gw, W;
    // sigma of (vertex, root); q = (1 + delta) / sigma once the vertex's delta is
    // final (a split row first accumulates its chunks' sums there); BFS level
    __device__ double *sg(int grp) const { return a.sg + (size_t)grp * n * G; }
    __device__ double *qq(int grp) const { return a.q + (size_t)grp * n * G; }
    __device__ uint8_t *lv(int grp) const { return a.lv + (size_t)grp * n * G; }
    __device__ Mk *vis(int grp) const { return reinterpret_cast<Mk *>(a.vis) + (size_t)grp * n; }
    // level masks: nm(grp, j)[v] = roots with v at level j (array j % 3)
    __device__ Mk *nm(int grp, int j) const { return reinterpret_cast<Mk *>(a.nm) + ((size_t)grp * 3 + (j % 3)) * n; }
    __device__ int32_t *vq(int grp) const { return a.vq + (size_t)grp * a.vcap; }
    __device__ Mk *vm(int grp) const { return reinterpret_cast<Mk *>(a.vm) + (size_t)grp * a.vcap; }
    __device__ int2 *tq(int grp) const { return a.tq + (size_t)grp * a.tcap; }
    __device__ int32_t *toff(int grp) const { return a.toff + (size_t)grp * (kMsMaxLev + 3); }
    __device__ MsGroup *ctr(int grp) const { return reinterpret_cast<MsGroup *>(a.ctr) + grp; }
    // root-major state index of root b of group grp
    __device__ size_t st(int grp, int b, int v) const { return (size_t)((a.g0 + grp) * G + b) * n + v; }

    // append w (first claimer) to the next level: its vertex entry and its row chunks
    __device__ void append(int grp, int w) const {
        const int2 r = full_row(a.g, w);
        const int deg = r.y - r.x;
        const int nch = deg > a.chunk ? (deg + a.chunk - 1) / a.chunk : 1;
        MsGroup *c = ctr(grp);
        const int vi = atomicAdd(&c->vcount, 1);
        const int ti = atomicAdd(&c->tcount, nch);
        if (vi >= a.vcap || (int64_t)ti + nch > a.tcap) {
            c->overflow = 1;
            return;
        }
        vq(grp)[vi] = w;
        int2 *t = tq(grp) + ti;
        for (int k = 0; k < nch; ++k) t[k] = make_int2(vi, k);
    }
};

// A pass's tasks over all groups of the wave: s_pref = prefix of the
// per-group task counts, s_lo = first task of each group's level.  Group of
// task t: the largest g with s_pref[g] <= t.
__device__ __forceinline__ int group_of(const int *s_pref, int ng, int t) {
    int lo = 0, hi = ng - 1;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (s_pref[mid] <= t) lo = mid; else hi = mid - 1;
    }
    return lo;
}

// Lane i's task of the warp's batch of 32; off = exclusive prefix of the
// chunk lengths (entry e of the batch belongs to the largest i with off_i <= e).
template <class Mk>
struct Task {
    int grp, vi, w, chunk, deg, beg, len, off;
    Mk m;
    bool valid;
};

template <int R>
__device__ __forceinline__ Task<typename MaskOf<R>::T> load_task(const Ms<R> &M, const int *s_pref, const int *s_lo,
                                                                 int ng, int t, int total, int T) {
    Task<typename MaskOf<R>::T> k{};
    k.valid = t < total;
    if (k.valid) {
        k.grp = group_of(s_pref, ng, t);
        const int2 tk = __ldcg(M.tq(k.grp) + s_lo[k.grp] + t - s_pref[k.grp]);
        k.vi = tk.x;
        k.chunk = tk.y;
        k.w = __ldcg(M.vq(k.grp) + tk.x);
        const int2 r = full_row(M.a.g, k.w);
        k.deg = r.y - r.x;
        k.beg = r.x + k.chunk * T;
        k.len = max(0, min(r.y, k.beg + T) - k.beg);
    }
    return k;
}

template <class Tk>
__device__ __forceinline__ int scan_len(Tk &k, int lane) {
    int x = k.len;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const int y = __shfl_up_sync(kFull, x, d);
        if (lane >= d) x += y;
    }
    k.off = x - k.len;
    return __shfl_sync(kFull, x, 31);
}

__device__ __forceinline__ int task_of(int off, int e) {
    int i = 0;
#pragma unroll
    for (int step = 16; step > 0; step >>= 1) {
        const int o = __shfl_sync(kFull, off, i + step);
        if (o <= e) i += step;
    }
    return i;
}

// Block-wide: s_lo / s_pref over the groups for the tasks toff[j] .. toff[j+1].
template <class MsT>
__device__ __forceinline__ void level_tasks(const MsT &M, int ng, int j, int *s_pref, int *s_lo) {
    if (threadIdx.x < ng) {
        const int *to = M.toff(threadIdx.x);
        s_lo[threadIdx.x] = __ldcg(to + j);
        s_pref[threadIdx.x + 1] = __ldcg(to + j + 1) - __ldcg(to + j);
    } else if (threadIdx.x == ng) {
        s_pref[0] = 0;
    }
    __syncthreads();
    if (threadIdx.x == 0)
        for (int i = 0; i < ng; ++i) s_pref[i + 1] += s_pref[i];
    __syncthreads();
}

// nm(j)[v] = 0 for the vertices of level j (their chunk-0 tasks), all groups.
template <class MsT>
__device__ __forceinline__ void clear_level(const MsT &M, int ng, int j) {
    if (j < 0) return;
    const int tid = blockIdx.x * kMsThreads + threadIdx.x;
    const int nth = gridDim.x * kMsThreads;
    for (int grp = 0; grp < ng; ++grp) {
        const int lo = __ldcg(M.toff(grp) + j), hi = __ldcg(M.toff(grp) + j + 1);
        auto *nm = M.nm(grp, j);
        for (int t = lo + tid; t < hi; t += nth) {
            const int2 tk = __ldcg(M.tq(grp) + t);
            if (tk.y == 0) nm[__ldcg(M.vq(grp) + tk.x)] = 0;
        }
    }
}

__device__ __forceinline__ double warp_sum(double x) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) x += __shfl_xor_sync(kFull, x, off);
    return x;
}

template <int R>
__global__ void __launch_bounds__(kMsThreads, 3) ms_kernel(MsArgs a) {
    using Mk = typename MaskOf<R>::T;
    constexpr int G = 32 * R;
    constexpr int U = kMsUnroll / R;  // contributing entries in flight (R gathers each)
    __shared__ int s_pref[kMsMaxG + 1];
    __shared__ int s_lo[kMsMaxG];
    __shared__ int s_done;
    __shared__ int s_d[G][33];
    __shared__ double s_sd[2][G][33];
    Ms<R> M{a, (size_t)a.n, (int)(threadIdx.x & 31), (int)((blockIdx.x * kMsThreads + threadIdx.x) >> 5),
            (int)((gridDim.x * kMsThreads) >> 5)};
    const int lane = M.lane;
    const int ng = a.ng;
    const GView &g = a.g;
    const int T = a.chunk;
    const size_t n = M.n;
    unsigned long long bytes = 0;  // algorithmic bytes (SURVEY.md Sec. 8(d) model)

    // ---- level 0: the roots (one warp per group)
    if (M.gw < ng) {
        const int grp = M.gw;
#pragma unroll
        for (int j = 0; j < R; ++j) {
            const int b = lane + 32 * j;
            const int slot = (a.g0 + grp) * G + b;
            if (slot < a.k_loc) {  // roots are distinct (dbc_create)
                const int s = a.roots[slot];
                M.sg(grp)[(size_t)s * G + b] = 1.0;
                M.lv(grp)[(size_t)s * G + b] = 0;
                const Mk mb = (Mk)1 << b;
                const int vi = atomicAdd(&M.ctr(grp)->vcount, 1);
                M.vq(grp)[vi] = s;
                M.vm(grp)[vi] = mb;
                M.vis(grp)[s] = mb;
                M.nm(grp, 0)[s] = mb;
                const int2 r = full_row(g, s);
                const int deg = r.y - r.x;
                const int nch = deg > T ? (deg + T - 1) / T : 1;
                const int ti = atomicAdd(&M.ctr(grp)->tcount, nch);
                for (int k = 0; k < nch; ++k) M.tq(grp)[ti + k] = make_int2(vi, k);
            }
        }
        __syncwarp();
        if (lane == 0) {
            M.toff(grp)[0] = 0;
            M.toff(grp)[1] = __ldcg(&M.ctr(grp)->tcount);
        }
    }
    grid_sync(a.bar);
    ms_trace(a.stats, 1, 0);

    int L = 0;
    for (;; ++L) {
        // ---- pass A: expand level L (tasks toff[L] .. toff[L+1])
        level_tasks(M, ng, L, s_pref, s_lo);
        for (int t0 = M.gw * 32; t0 < s_pref[ng]; t0 += M.W * 32) {
            auto k = load_task(M, s_pref, s_lo, ng, t0 + lane, s_pref[ng], T);
            if (k.valid) k.m = __ldcg(M.vm(k.grp) + k.vi);
            // sigma of a split row (chunk partials added atomically): exact below
            // 2^53; at or above it, re-summed in canonical order; then stored
            uint32_t fix = __ballot_sync(kFull, k.valid && k.chunk == 0 && k.deg > T && L > 0);
            while (fix) {
                const int i = __ffs(fix) - 1;
                fix &= fix - 1;
                const int grp = __shfl_sync(kFull, k.grp, i), u = __shfl_sync(kFull, k.w, i);
                const Mk mu = __shfl_sync(kFull, k.m, i);
                double sum[R];
                bool big[R], anyb = false;
#pragma unroll
                for (int j = 0; j < R; ++j) {
                    const int b = lane + 32 * j;
                    sum[j] = bit(mu, b) ? __ldcg(M.sg(grp) + (size_t)u * G + b) : 0.0;
                    big[j] = bit(mu, b) && sum[j] >= kExact;
                    anyb |= big[j];
                }
                if (__any_sync(kFull, anyb)) {
                    const int2 r = full_row(g, u);
                    const Mk *pm = M.nm(grp, L - 1);
                    double s2[R] = {};
                    for (int jj = r.x; jj < r.y; ++jj) {
                        const int x = ldg_i(g.col + jj);
                        const Mk px = anyb ? __ldcg(pm + x) : (Mk)0;
#pragma unroll
                        for (int j = 0; j < R; ++j)
                            if (big[j] && bit(px, lane + 32 * j))
                                s2[j] += __ldcg(M.sg(grp) + (size_t)x * G + lane + 32 * j);
                    }
#pragma unroll
                    for (int j = 0; j < R; ++j)
                        if (big[j]) {
                            sum[j] = s2[j];
                            M.sg(grp)[(size_t)u * G + lane + 32 * j] = sum[j];
                        }
                }
            }
            const int E = scan_len(k, lane);
            for (int base = 0; base < E; base += 32) {
                const int e = base + lane;
                const int i = task_of(k.off, e);
                const int gi = __shfl_sync(kFull, k.grp, i), bi = __shfl_sync(kFull, k.beg, i);
                const int oi = __shfl_sync(kFull, k.off, i);
                const Mk mi = __shfl_sync(kFull, k.m, i);
                if (e < E) {
                    const int w = ldg_i(g.col + bi + e - oi);
                    const Mk nmk = mi & ~__ldcg(M.vis(gi) + w);
                    if (nmk) {
                        const Mk old = atomicOr(M.nm(gi, L + 1) + w, nmk);
                        if (old == 0) M.append(gi, w);
                    }
                }
            }
        }
        grid_sync(a.bar);
        ms_trace(a.stats, 2, L);

        // ---- level L+1: tasks toff[L+1] .. tcount (stable until the next pass A)
        const int Lc = L + 1;
        if (threadIdx.x < ng) {
            const int grp = threadIdx.x;
            const int lo = __ldcg(M.toff(grp) + Lc);
            const int hi = min(__ldcg(&M.ctr(grp)->tcount), (int)a.tcap);
            s_lo[grp] = lo;
            s_pref[grp + 1] = hi - lo;
            if (blockIdx.x == 0) M.toff(grp)[Lc + 1] = hi;
        } else if (threadIdx.x == ng) {
            s_pref[0] = 0;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            for (int i = 0; i < ng; ++i) s_pref[i + 1] += s_pref[i];
            int ovf = 0;
            for (int i = 0; i < ng; ++i) ovf |= __ldcg(&M.ctr(i)->overflow);
            s_done = (s_pref[ng] == 0) ? 1 : (ovf || Lc > kMsMaxLev) ? 2 : 0;
        }
        __syncthreads();
        if (s_done) {
            if (s_done == 2 && blockIdx.x == 0 && threadIdx.x == 0) M.ctr(0)->overflow = 1;
            break;
        }
        // ---- pass B: sigma pull of level Lc from level L (canonical order)
        clear_level(M, ng, Lc - 2);  // nm(Lc - 2) is pass A(Lc)'s discovery array
        for (int t0 = M.gw * 32; t0 < s_pref[ng]; t0 += M.W * 32) {
            auto k = load_task(M, s_pref, s_lo, ng, t0 + lane, s_pref[ng], T);
            if (k.valid) {
                k.m = __ldcg(M.nm(k.grp, Lc) + k.w);
                bytes += (unsigned long long)popc_m(k.m) * 8ull * k.len;  // col + d per entry
                if (k.chunk == 0) {  // the vertex's level-Lc record
                    M.vm(k.grp)[k.vi] = k.m;
                    M.vis(k.grp)[k.w] = __ldcg(M.vis(k.grp) + k.w) | k.m;
                    uint4 *lp = reinterpret_cast<uint4 *>(M.lv(k.grp) + (size_t)k.w * G);
                    const uint32_t rep = (uint32_t)Lc * 0x01010101u;
#pragma unroll
                    for (int h = 0; h < 2 * R; ++h) {  // 16 roots per uint4: their bytes := Lc
                        uint4 q4 = __ldcg(lp + h);
                        uint32_t *wd = reinterpret_cast<uint32_t *>(&q4);
#pragma unroll
                        for (int j = 0; j < 4; ++j) {
                            const uint32_t nib = (uint32_t)(k.m >> (16 * h + 4 * j)) & 0xFu;
                            const uint32_t bm = ((nib & 1u) ? 0xFFu : 0u) | ((nib & 2u) ? 0xFF00u : 0u) |
                                                ((nib & 4u) ? 0xFF0000u : 0u) | ((nib & 8u) ? 0xFF000000u : 0u);
                            wd[j] = (wd[j] & ~bm) | (rep & bm);
                        }
                        if ((k.m >> (16 * h)) & 0xFFFFu) lp[h] = q4;
                    }
                    bytes += (unsigned long long)popc_m(k.m) * (16 + 4);  // row bounds, sigma and d writes
                }
            }
            const int E = scan_len(k, lane);
            int cur = -1;
            double sum[R];
            auto flush = [&]() {  // sigma of task cur (uniform)
                const int gc = __shfl_sync(kFull, k.grp, cur), wc = __shfl_sync(kFull, k.w, cur);
                const Mk mc = __shfl_sync(kFull, k.m, cur);
                const bool split = __shfl_sync(kFull, k.deg, cur) > T;
#pragma unroll
                for (int j = 0; j < R; ++j) {
                    const int b = lane + 32 * j;
                    if (bit(mc, b)) {
                        double *sw = M.sg(gc) + (size_t)wc * G + b;
                        if (split)
                            atomicAdd(sw, sum[j]);
                        else
                            *sw = sum[j];
                        if (!(sum[j] <= 1.7976931348623157e308)) atomicOr(a.err, kErrNumeric);
                    }
                }
            };
            for (int base = 0; base < E; base += 32) {
                const int e = base + lane;
                const int i = task_of(k.off, e);
                const int gi = __shfl_sync(kFull, k.grp, i), bi = __shfl_sync(kFull, k.beg, i);
                const int oi = __shfl_sync(kFull, k.off, i);
                const Mk mi = __shfl_sync(kFull, k.m, i);
                const int x = e < E ? ldg_i(g.col + bi + e - oi) : 0;
                const Mk pm = e < E ? (__ldcg(M.nm(gi, L) + x) & mi) : (Mk)0;
                bytes += 8ull * popc_m(pm);  // sigma of a predecessor (per root)
                uint32_t todo = __ballot_sync(kFull, pm != 0);
                while (todo) {
                    int ts[U];
                    Mk bits[U];
                    double sx[U][R];
#pragma unroll
                    for (int q = 0; q < U; ++q) {
                        const int kk = __ffs(todo) - 1;  // -1: past the last one
                        todo &= todo - 1;
                        const int xs = __shfl_sync(kFull, x, kk & 31);
                        const int gs = __shfl_sync(kFull, gi, kk & 31);
                        ts[q] = kk < 0 ? -1 : __shfl_sync(kFull, i, kk & 31);
                        bits[q] = kk < 0 ? (Mk)0 : __shfl_sync(kFull, pm, kk & 31);
                        const double *sp = M.sg(gs) + (size_t)xs * G + lane;
#pragma unroll
                        for (int j = 0; j < R; ++j) sx[q][j] = bit(bits[q], lane + 32 * j) ? __ldcg(sp + 32 * j) : 0.0;
                    }
#pragma unroll
                    for (int q = 0; q < U; ++q) {
                        if (ts[q] < 0) break;
                        if (ts[q] != cur) {
                            if (cur >= 0) flush();
                            cur = ts[q];
#pragma unroll
                            for (int j = 0; j < R; ++j) sum[j] = 0.0;
                        }
#pragma unroll
                        for (int j = 0; j < R; ++j)
                            if (bit(bits[q], lane + 32 * j)) sum[j] += sx[q][j];
                    }
                }
            }
            if (cur >= 0) flush();
        }
        grid_sync(a.bar);
        ms_trace(a.stats, 3, Lc);
    }
    const int maxlev = L;  // levels 0 .. maxlev are non-empty (some group)

    // ---- backward, Eq. (2): delta(w) = sigma(w) * sum over successors y of
    // q(y), q(y) = (1 + delta(y)) / sigma(y).  nm(j) holds level j's masks
    // again: pass Lc reads nm(Lc + 1), scatters level Lc into nm(Lc) for pass
    // Lc - 1 and clears level Lc + 2 from nm(Lc + 2).  (The forward loop leaves
    // nm(maxlev) and nm(maxlev - 1) exact and the third array clean.)  The
    // deepest level is a pass too: no successors, but its q = 1 / sigma.
    for (int Lc = maxlev; Lc >= 1; --Lc) {
        level_tasks(M, ng, Lc, s_pref, s_lo);
        if (Lc + 2 <= maxlev) clear_level(M, ng, Lc + 2);
        for (int t0 = M.gw * 32; t0 < s_pref[ng]; t0 += M.W * 32) {
            auto k = load_task(M, s_pref, s_lo, ng, t0 + lane, s_pref[ng], T);
            if (k.valid) {
                k.m = __ldcg(M.vm(k.grp) + k.vi);
                if (k.chunk == 0) M.nm(k.grp, Lc)[k.w] = k.m;
                bytes += (unsigned long long)popc_m(k.m) * (8ull * k.len + (k.chunk == 0 ? 48 : 0));
            }
            const int E = scan_len(k, lane);
            int cur = -1;
            uint32_t seen = 0;  // tasks of the batch that had successors
            double acc[R], sv[R];
            auto flush = [&]() {  // delta (and q) of task cur (uniform)
                const int gc = __shfl_sync(kFull, k.grp, cur), wc = __shfl_sync(kFull, k.w, cur);
                const Mk mc = __shfl_sync(kFull, k.m, cur);
                const bool split = __shfl_sync(kFull, k.deg, cur) > T;
                double bsum = 0.0;
#pragma unroll
                for (int j = 0; j < R; ++j) {
                    const int b = lane + 32 * j;
                    const bool act = bit(mc, b);
                    if (split) {  // a chunk's sum: q and BC once the pass is over
                        if (act && acc[j] != 0.0) atomicAdd(M.qq(gc) + (size_t)wc * G + b, acc[j]);
                    } else if (act) {
                        const double dl = __dmul_rn(sv[j], acc[j]);
                        M.qq(gc)[(size_t)wc * G + b] = __ddiv_rn(__dadd_rn(1.0, dl), sv[j]);
                        bsum += dl;
                    }
                }
                if (!split) {
                    bsum = warp_sum(bsum);
                    if (lane == 0 && bsum != 0.0) atomicAdd(a.bc + wc, bsum);
                }
            };
            auto begin = [&](int c) {  // task c becomes current: prefetch its sigma
                cur = c;
                seen |= 1u << c;
                const int gc = __shfl_sync(kFull, k.grp, c), wc = __shfl_sync(kFull, k.w, c);
                const Mk mc = __shfl_sync(kFull, k.m, c);
#pragma unroll
                for (int j = 0; j < R; ++j) {
                    acc[j] = 0.0;
                    // sigma is read-only in the backward passes (L1-cached loads)
                    sv[j] = bit(mc, lane + 32 * j) ? M.sg(gc)[(size_t)wc * G + lane + 32 * j] : 1.0;
                }
            };
            for (int base = 0; base < E; base += 32) {
                const int e = base + lane;
                const int i = task_of(k.off, e);
                const int gi = __shfl_sync(kFull, k.grp, i), bi = __shfl_sync(kFull, k.beg, i);
                const int oi = __shfl_sync(kFull, k.off, i);
                const Mk mi = __shfl_sync(kFull, k.m, i);
                const int y = e < E ? ldg_i(g.col + bi + e - oi) : 0;
                const Mk pm = e < E ? (__ldcg(M.nm(gi, Lc + 1) + y) & mi) : (Mk)0;
                bytes += 16ull * popc_m(pm);  // sigma, delta of a successor (per root)
                uint32_t todo = __ballot_sync(kFull, pm != 0);
                while (todo) {
                    int ts[U];
                    Mk bits[U];
                    double qy[U][R];
#pragma unroll
                    for (int q = 0; q < U; ++q) {
                        const int kk = __ffs(todo) - 1;
                        todo &= todo - 1;
                        const int ys = __shfl_sync(kFull, y, kk & 31);
                        const int gs = __shfl_sync(kFull, gi, kk & 31);
                        ts[q] = kk < 0 ? -1 : __shfl_sync(kFull, i, kk & 31);
                        bits[q] = kk < 0 ? (Mk)0 : __shfl_sync(kFull, pm, kk & 31);
                        const double *qp = M.qq(gs) + (size_t)ys * G + lane;
#pragma unroll
                        for (int j = 0; j < R; ++j) qy[q][j] = bit(bits[q], lane + 32 * j) ? __ldcg(qp + 32 * j) : 0.0;
                    }
#pragma unroll
                    for (int q = 0; q < U; ++q) {
                        if (ts[q] < 0) break;
                        if (ts[q] != cur) {
                            if (cur >= 0) flush();
                            begin(ts[q]);
                        }
#pragma unroll
                        for (int j = 0; j < R; ++j)
                            if (bit(bits[q], lane + 32 * j)) acc[j] += qy[q][j];
                    }
                }
            }
            if (cur >= 0) flush();
            // whole (unsplit) rows without successors in any lane: delta 0, q = 1 / sigma
            uint32_t rest = __ballot_sync(kFull, k.valid && k.deg <= T) & ~seen;
            while (rest) {
                const int c = __ffs(rest) - 1;
                rest &= rest - 1;
                begin(c);
                flush();
            }
        }
        grid_sync(a.bar);
        // split rows of level Lc: delta is final now -> q and BC
        for (int t0 = M.gw * 32; t0 < s_pref[ng]; t0 += M.W * 32) {
            const int t = t0 + lane;
            bool sp = false;
            int grp = 0, w = 0;
            Mk m = 0;
            if (t < s_pref[ng]) {
                grp = group_of(s_pref, ng, t);
                const int2 tk = __ldcg(M.tq(grp) + s_lo[grp] + t - s_pref[grp]);
                if (tk.y == 0) {
                    w = __ldcg(M.vq(grp) + tk.x);
                    const int2 r = full_row(g, w);
                    if (r.y - r.x > T) {
                        sp = true;
                        m = __ldcg(M.vm(grp) + tk.x);
                    }
                }
            }
            uint32_t todo = __ballot_sync(kFull, sp);
            while (todo) {
                const int i = __ffs(todo) - 1;
                todo &= todo - 1;
                const int gc = __shfl_sync(kFull, grp, i), wc = __shfl_sync(kFull, w, i);
                const Mk mc = __shfl_sync(kFull, m, i);
                double bsum = 0.0;
#pragma unroll
                for (int j = 0; j < R; ++j) {
                    const int b = lane + 32 * j;
                    if (bit(mc, b)) {
                        double *q = M.qq(gc) + (size_t)wc * G + b;
                        const double sw = M.sg(gc)[(size_t)wc * G + b];
                        const double dl = __dmul_rn(sw, __ldcg(q));
                        *q = __ddiv_rn(__dadd_rn(1.0, dl), sw);
                        bsum += dl;
                    }
                }
                bsum = warp_sum(bsum);
                if (lane == 0 && bsum != 0.0) atomicAdd(a.bc + wc, bsum);
            }
        }
        grid_sync(a.bar);
        ms_trace(a.stats, 4, Lc);
    }

    // ---- the root-major state of the dynamic kernels (Alg. 1's d, sigma,
    // delta): tiles of 32 vertices x G roots through shared memory, so both
    // the vertex-major reads and the root-major writes are coalesced;
    // delta = q sigma - 1 (q = (1 + delta) / sigma: within 2^-51 relative, floor 1)
    {
        const int warp = threadIdx.x >> 5;
        const size_t ntile = (n + 31) / 32;
        for (size_t tile = blockIdx.x; tile < ntile * (size_t)ng; tile += gridDim.x) {
            const int grp = (int)(tile / ntile);
            const size_t v0 = (tile % ntile) * 32;
            for (int i = warp; i < 32; i += kMsThreads / 32) {  // warp: vertex v0 + i, lane: roots
                const size_t v = v0 + i;
                if (v >= n) break;
#pragma unroll
                for (int j = 0; j < R; ++j) {
                    const int b = lane + 32 * j;
                    const size_t o = v * G + b;
                    const int l = __ldcg(M.lv(grp) + o);
                    const double sw = l == 255 ? 0.0 : __ldcg(M.sg(grp) + o);
                    const double dl = (l == 255 || l == 0) ? 0.0 : __dsub_rn(__dmul_rn(__ldcg(M.qq(grp) + o), sw), 1.0);
                    s_d[b][i] = l == 255 ? kInf : l;
                    s_sd[0][b][i] = sw;
                    s_sd[1][b][i] = dl;
                }
            }
            __syncthreads();
            const int s0 = (a.g0 + grp) * G;
            for (int b = warp; b < G; b += kMsThreads / 32) {  // warp: root b, lane: vertex
                const size_t v = v0 + lane;
                if (s0 + b < a.k_loc && v < n) {
                    a.d[(size_t)(s0 + b) * n + v] = s_d[b][lane];
                    a.sd[(size_t)(s0 + b) * n + v] = make_double2(s_sd[0][b][lane], s_sd[1][b][lane]);
                }
            }
            __syncthreads();
        }
        if (blockIdx.x == 0 && threadIdx.x == 0) bytes += 20ull * (size_t)max(0, min(a.k_loc - a.g0 * G, ng * G)) * n;
    }

#pragma unroll
    for (int off = 16; off > 0; off >>= 1) bytes += __shfl_xor_sync(kFull, bytes, off);
    if (lane == 0 && bytes) atomicAdd(stat_lane(a.stats) + kStStaticBytes, bytes);
}

// Level-2 predecessor masks of roots with at most kMaskDeg neighbours (read by
// the update kernels' level-2 shortcut), from the root-major state.
__global__ void __launch_bounds__(kBlock) ms_l2mask_kernel(StaticArgs a) {
    const int slot = blockIdx.x;
    const size_t n = (size_t)a.n;
    const int s = a.roots[slot];
    const Root st{a.d + (size_t)slot * n, a.sd + (size_t)slot * n};
    const int2 rs = full_row(a.g, s);
    const bool ok = rs.y - rs.x <= kMaskDeg;
    if (ok) build_l2masks(a.g, st, a.l2mask + (size_t)slot * n, rs, INT32_MAX);
    if (threadIdx.x == 0) a.mask_ds[slot] = ok ? rs.y - rs.x : -1;
}

}  // namespace

int ms_static_max_groups() { return kMsMaxG; }
int ms_static_max_levels() { return kMsMaxLev; }
size_t ms_static_counter_bytes(int ng) { return sizeof(MsGroup) * (size_t)ng; }

int ms_static_resident(int nsm, int r) {
    int per = 0;
    const void *k = r == 2 ? (const void *)ms_kernel<2> : (const void *)ms_kernel<1>;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k, kMsThreads, 0) != cudaSuccess) return 0;
    return per * nsm;
}

cudaError_t launch_static_ms(const MsArgs &a, int r, int grid, cudaStream_t s) {
    MsArgs copy = a;
    void *args[] = {&copy};
    const void *k = r == 2 ? (const void *)ms_kernel<2> : (const void *)ms_kernel<1>;
    return cudaLaunchCooperativeKernel(k, dim3(grid), dim3(kMsThreads), args, 0, s);
}

void launch_static_l2mask(const StaticArgs &a, cudaStream_t s) {
    if (a.k_loc > 0) ms_l2mask_kernel<<<a.k_loc, kBlock, 0, s>>>(a);
}

}  // namespace dbc
