// cube.cu — dense MOLAP cube in B200 HBM and the batched sub-cube range-reduce.
//
// Hot path per batch:
//   plan_kernel      a1/a3/a4/a5  per query: validate, intersect with the shard,
//                    linearise the box into runs (Fig. 2 "area of limited search",
//                    PAPER.md:143,151), size work units and items, scan -> item table
//   reduce_kernel    a6/a7        persistent grid, items popped from a device
//                    counter; streams runs with 128-bit / 32-bit loads; per-item
//                    partials, fixed-order per-query combine by the last block
//   finalize_kernel  a9           COUNT = V (Eq. 3), AVG = SUM/V, flags
// The per-query partial format (olap.h) is what crosses GPUs (a8).
#include <algorithm>
#include <climits>
#include <cstdlib>
#include <cstring>
#include <atomic>
#include <mutex>
#include <new>
#include <type_traits>
#include <vector>

#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include "common.cuh"
#include "mgpu.h"

namespace olap {

constexpr int kMaxDims = 8;
constexpr int kMaxRunDims = 7;
constexpr int kWarps = 8;                   // warps per reduce block
constexpr int kThreads = kWarps * 32;
constexpr int kTaskSlots = 2048;            // slots per warp task (long path), slot budget of a short task
constexpr int kShortMaxSlots = 512;         // runs of at most this many slots: short path (<= 31 runs per task)
#ifndef OLAP_UNROLL
#define OLAP_UNROLL 4
#endif
constexpr int kUnroll = OLAP_UNROLL;        // independent loads in flight per lane
#ifndef OLAP_MIN_BLOCKS
#define OLAP_MIN_BLOCKS 4
#endif
constexpr int kMinBlocks = OLAP_MIN_BLOCKS;
#ifndef OLAP_WARP_ITEMS
#define OLAP_WARP_ITEMS -1
#endif
// Item granularity: block items (reduce_kernel: 8 warps share an item) or warp items
// (reduce_kernel_w: no block barriers).  -1 = per batch: warp items when the batch has more
// than kWarpItemQueries queries per resident block (many small boxes: C5, bricked
// sub-boxes; measured +13% there and -7% on C1's 1,000 queries); 0 / 1 force one.
constexpr int kWarpItemsMode = OLAP_WARP_ITEMS;
constexpr int64_t kWarpItemQueries = 8;
constexpr int64_t kItemCells = 262144;      // minimum item: 1 MiB of 4-byte cells
constexpr int64_t kMaxExtent = (1ll << 30); // per-dimension limit (32-bit digit arithmetic)
constexpr int64_t kMaxCells = (1ll << 42);
constexpr int64_t kGraphMaxQueries = 16384;  // olap_query_batch replays CUDA graphs up to this batch size

// op class of a query: which accumulator the hot loop keeps (SUM and AVG share one)
enum : int32_t { OPC_NONE = 0, OPC_SUM = 1, OPC_MIN = 2, OPC_MAX = 3 };

// Per-query plan (shard-local).  The box is R runs of L consecutive cells (all dims
// after the split dim k are full and merge into the run, Fig. 2 / DESIGN.md "runs").
// Run r starts at cell  base + sum_e digit_e(r) * rs[e]  (digits of r in radix
// frl[e].d, innermost first).  When every run stride is a multiple of 4 cells all runs
// share the same 16-B misalignment h0, so each run is covered by nslot aligned 16-B
// "slots" (V = 4 cells) whose first h0 and trailing cells are masked; otherwise V = 1.
// Slots of all runs are flattened (G = R * nslot) and cut into warp tasks of T slots.
struct QDesc {
    int64_t base_al;  // first slot of run 0 (cells, multiple of V)
    int64_t L;        // run length (cells)
    int64_t R;        // number of runs
    int64_t nslot;    // slots per run
    int64_t G;        // slots in the box
    int64_t tasks;    // ceil(G / T)
    int64_t vlocal;   // cells of the box on this shard (R * L)
    int32_t T;        // short path: runs per task (<= 31); long path: slots per task
    int32_t tpi;      // tasks per item
    int32_t h0;       // masked leading cells of each run's first slot
    int32_t V;        // cells per slot (8, 4 or 1)
    int32_t opc, nrd, op, shortp;  // shortp: runs of <= kShortMaxSlots slots take the short path
    FastDiv fnslot;   // / nslot (long path; valid when nslot < 2^31)
    FastDiv fni;      // / (nslot - 2), the interior slots of a run (short path)
    FastDiv frl[kMaxRunDims];
    int64_t rs[kMaxRunDims];
};

struct Geo {
    int nd, dtype;
    int64_t G, g, b;
    int64_t n[kMaxDims];       // global extents
    int64_t stride[kMaxDims];  // local strides (cells; the innermost pitch may be padded)
    int64_t local_rows;
    int64_t pitch;             // cells per innermost row in HBM (n[nd-1] rounded up to 4 when padded)
    int64_t lrow;              // logical (unpadded) cells per dim-0 row
    int padded;                // pitch != n[nd-1]: runs never merge across innermost rows
};

struct Extents {
    int64_t n[kMaxDims];
};

// ------------------------------------------------------------------ device helpers

// Cube loads use ld.global.nc (L1-allocating).  Measured +9-10% over L1::no_allocate on
// C2a/C3/C4 once the data is L2-resident (profiles/sweep_r01_load_flavor.txt) although the
// L1 hit rate stays ~2% (ncu): the no_allocate variant costs more L1TEX pipeline
// throughput (80% vs 73% at the same work), which is what bounds the L2-served kernel.
#ifndef OLAP_LD4
#define OLAP_LD4 "ld.global.nc.v4.u32"
#endif
#ifndef OLAP_LD1
#define OLAP_LD1 "ld.global.nc.u32"
#endif
__device__ __forceinline__ uint4 ld_stream4(const void* p) {
    uint4 r;
    asm(OLAP_LD4 " {%0,%1,%2,%3}, [%4];"
        : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
        : "l"(p));
    return r;
}
#ifndef OLAP_LD8
#define OLAP_LD8 "ld.global.nc.v8.u32"
#endif
__device__ __forceinline__ void ld_stream8(const void* p, uint32_t (&r)[8]) {  // LDG.256 (sm_100)
    asm(OLAP_LD8 " {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
        : "l"(p));
}
__device__ __forceinline__ uint32_t ld_stream1(const void* p) {
    uint32_t r;
    asm(OLAP_LD1 " %0, [%1];" : "=r"(r) : "l"(p));
    return r;
}

__device__ __forceinline__ int32_t f32_code(float f) {
    int32_t b = __float_as_int(f);
    return b ^ ((b >> 31) & 0x7fffffff);
}
__host__ __device__ __forceinline__ float f32_decode(int32_t c) {
    int32_t b = c ^ ((c >> 31) & 0x7fffffff);
#ifdef __CUDA_ARCH__
    return __int_as_float(b);
#else
    float f;
    std::memcpy(&f, &b, 4);
    return f;
#endif
}

__device__ __forceinline__ FastDiv dev_fastdiv(uint32_t d) {
    FastDiv f;
    f.d = d;
    f.l = d <= 1 ? 0u : 32u - __clz(d - 1);  // ceil(log2 d)
    f.m = (uint32_t)(((1ull << 32) * ((1ull << f.l) - d)) / d + 1);
    return f;
}

// Per-lane accumulators.  int32 cells: SUM in uint64 (wraparound, reading R7),
// MIN/MAX in int32.  float32 cells: SUM in double (reading R8), MIN/MAX in float.
// add<OPC>(bits, mk): mk is an all-ones / all-zero mask of the cell; a masked cell
// contributes the op's identity through one LOP3 on the raw bits (0 -> +0.0 / 0 for
// SUM, +inf / INT_MAX for MIN, -inf / INT_MIN for MAX), so no select on the result.
// int32 SUM accumulates the biased cells u = v + 2^31 (= v ^ 0x80000000, an unsigned 32-bit
// value: no sign extension; the masking LOP3 applies the bias too, and two cells go into one
// 64-bit IADD3 / IADD3.X pair) and subtracts nb * 2^31 at the end: the same sum mod 2^64
// (reading R7).  Measured: C4 110.5k -> 124.7k q/s, C1 +4%.
struct AccI {
    unsigned long long s;
    uint32_t nb;  // cells folded into s (each carried a 2^31 bias)
    int32_t mn, mx;
    __device__ void init() { s = 0ull; nb = 0u; mn = INT_MAX; mx = INT_MIN; }
    template <int OPC>
    __device__ __forceinline__ void add(uint32_t bits, uint32_t mk) {
        if (OPC == OPC_SUM) {
            s += (unsigned long long)((bits & mk) ^ 0x80000000u);
            ++nb;
        }
        if (OPC == OPC_MIN) mn = min(mn, (int32_t)((bits & mk) | (0x7fffffffu & ~mk)));
        if (OPC == OPC_MAX) mx = max(mx, (int32_t)((bits & mk) | (0x80000000u & ~mk)));
    }
    __device__ __forceinline__ long long sum_bits() const { return (long long)(s - ((unsigned long long)nb << 31)); }
    __device__ __forceinline__ int32_t code_max() const { return mx; }
    __device__ __forceinline__ int32_t code_min() const { return mn; }
};
struct AccF {
    double s;
    float mn, mx;
    __device__ void init() { s = 0.0; mn = __int_as_float(0x7f800000); mx = __int_as_float(0xff800000); }
    template <int OPC>
    __device__ __forceinline__ void add(uint32_t bits, uint32_t mk) {
        if (OPC == OPC_SUM) s += (double)__uint_as_float(bits & mk);
        if (OPC == OPC_MIN) mn = fminf(mn, __uint_as_float((bits & mk) | (0x7f800000u & ~mk)));
        if (OPC == OPC_MAX) mx = fmaxf(mx, __uint_as_float((bits & mk) | (0xff800000u & ~mk)));
    }
    __device__ __forceinline__ long long sum_bits() const { return __double_as_longlong(s); }
    __device__ __forceinline__ int32_t code_max() const { return f32_code(mx); }
    __device__ __forceinline__ int32_t code_min() const { return f32_code(mn); }
};

template <class Acc> struct SumOps;
template <> struct SumOps<AccI> {
    __device__ static long long add(long long a, long long b) {
        return (long long)((unsigned long long)a + (unsigned long long)b);
    }
};
template <> struct SumOps<AccF> {
    __device__ static long long add(long long a, long long b) {
        return __double_as_longlong(__longlong_as_double(a) + __longlong_as_double(b));
    }
};

// First slot of run r: base_al + sum_e digit_e(r) * rs[e].  32-bit fast-division
// chain when r < 2^31 (the common case), 64-bit divisions otherwise.  The digit loop is
// deliberately not unrolled: the radices stay in shared memory instead of ~30 registers.
__device__ __noinline__ int64_t run_addr_wide(const QDesc& d, int64_t r) {  // r >= 2^31: rare
    int64_t a = d.base_al;
    for (int e = 0; e < d.nrd; ++e) {
        const int64_t l = d.frl[e].d, q = r / l;
        a += (r - q * l) * d.rs[e];
        r = q;
    }
    return a;
}

__device__ __forceinline__ int64_t run_addr(const QDesc& d, int64_t r) {
    if (r >= (1ll << 31)) return run_addr_wide(d, r);
    int64_t a = d.base_al;
    const int nrd = d.nrd;
    uint32_t x = (uint32_t)r;
#pragma unroll 1
    for (int e = 0; e < nrd; ++e) {
        const FastDiv f = d.frl[e];
        const uint32_t q = fdiv(x, f);
        a += (int64_t)(x - q * f.d) * d.rs[e];
        x = q;
    }
    return a;
}

// 64-bit quotient kept out of line (one per warp per item): no caller-saved spills in the loops
__device__ __noinline__ int64_t div64(int64_t a, int64_t b) { return a / b; }

// Largest q in [0,nq) with item_start[q] <= item (32-ary warp search).
__device__ __forceinline__ int64_t find_query(const int64_t* __restrict__ item_start, int64_t nq, int64_t item,
                                              int lane) {
    int64_t lo = 0, hi = nq;
    while (hi - lo > 32) {
        const int64_t step = (hi - lo + 31) / 32;
        const int64_t idx = lo + lane * step;
        const bool ok = idx < hi && __ldg(item_start + idx) <= item;
        const unsigned m = __ballot_sync(0xffffffffu, ok);
        const int l = 31 - __clz(m);
        lo = lo + l * step;
        hi = min(hi, lo + step);
    }
    const int64_t idx = lo + lane;
    const bool ok = idx < hi && __ldg(item_start + idx) <= item;
    const unsigned m = __ballot_sync(0xffffffffu, ok);
    return lo + (31 - __clz(m));
}

// Slot masks are byte-mask words: byte k = 0xFF when cell k of the slot is in the box
// (8 bytes for 8-cell slots).  Cell k's 32-bit mask is byte k replicated (one PRMT).
template <int V>
__device__ __forceinline__ uint32_t cell_mask(uint64_t w, int k) {
    if (V == 1) return (uint32_t)w;
    return __byte_perm(k < 4 ? (uint32_t)w : (uint32_t)(w >> 32), 0u, 0x1111u * (uint32_t)(k & 3));
}
__device__ __forceinline__ uint64_t byte_mask_word(uint32_t bits8) {
    uint64_t w = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k)
        if (bits8 >> k & 1u) w |= 0xFFull << (8 * k);
    return w;
}

// SM = true: p points into shared memory (the tile-shared scan stages cube tiles there);
// plain dereferences let the compiler emit LDS.128 (verified in SASS).  A 32-B slot is two
// LDS.128; lanes 4-7 of every 8 read the slot's upper half first, so each quarter-warp's
// first (and second) LDS.128 covers all 32 banks once instead of two-way conflicting on a
// 32-B lane stride.  Those lanes hold cells 4-7 in v[0..3]: sm_swap() swaps their masks.
__device__ __forceinline__ bool sm_swapped() { return (threadIdx.x >> 2) & 1; }
__device__ __forceinline__ uint32_t smem_addr_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
template <int V, bool SM = false>
__device__ __forceinline__ void load_slot(const uint32_t* p, uint32_t (&v)[V]) {
    if constexpr (SM) {
        if constexpr (V == 1) {
            v[0] = *p;
        } else if constexpr (V == 4) {
            const uint4 x = *reinterpret_cast<const uint4*>(p);
            v[0] = x.x;
            v[1] = x.y;
            v[2] = x.z;
            v[3] = x.w;
        } else {
            const int hf = sm_swapped() ? 4 : 0;
            const uint4 x = *reinterpret_cast<const uint4*>(p + hf);
            const uint4 y = *reinterpret_cast<const uint4*>(p + (4 - hf));
            v[0] = x.x;
            v[1] = x.y;
            v[2] = x.z;
            v[3] = x.w;
            v[4] = y.x;
            v[5] = y.y;
            v[6] = y.z;
            v[7] = y.w;
        }
    } else if constexpr (V == 8) {
        ld_stream8(p, v);
    } else if constexpr (V == 4) {
        const uint4 x = ld_stream4(p);
        v[0] = x.x;
        v[1] = x.y;
        v[2] = x.z;
        v[3] = x.w;
    } else {
        v[0] = ld_stream1(p);
    }
}

// Tile path (SM), float32 SUM: the cells of one slot are added pairwise in fp32 first (a
// tree of depth log2 V <= 3), then the slot sum joins the fp64 accumulator: one F2F + DADD
// per slot instead of per cell.  Each fp32 add rounds once (relative 2^-24), so a slot sum is
// off by at most 3 * 2^-24 * sum|x| and the query's SUM by at most ~1.8e-7 * sum|x| — within
// the 1e-6 tolerance (reading R8), and exact for integer-valued cells below
// 2^21 (every partial sum is an exact fp32).
template <int V>
__device__ __forceinline__ float slot_tree(const uint32_t (&x)[V]) {
    if constexpr (V == 8)
        return ((__uint_as_float(x[0]) + __uint_as_float(x[1])) + (__uint_as_float(x[2]) + __uint_as_float(x[3]))) +
               ((__uint_as_float(x[4]) + __uint_as_float(x[5])) + (__uint_as_float(x[6]) + __uint_as_float(x[7])));
    else if constexpr (V == 4)
        return (__uint_as_float(x[0]) + __uint_as_float(x[1])) + (__uint_as_float(x[2]) + __uint_as_float(x[3]));
    else
        return __uint_as_float(x[0]);
}
template <class Acc, int OPC, int V, bool SM>
constexpr bool tree_sum() {
    return SM && OPC == OPC_SUM && V >= 4 && std::is_same<Acc, AccF>::value;
}

template <class Acc, int OPC, int V, bool SM = false>
__device__ __forceinline__ void fold_slot(Acc& acc, const uint32_t (&v)[V], uint64_t w) {
    if (SM && V == 8 && sm_swapped()) w = (w >> 32) | (w << 32);
    if constexpr (tree_sum<Acc, OPC, V, SM>()) {
        uint32_t x[V];
#pragma unroll
        for (int k = 0; k < V; ++k) x[k] = v[k] & cell_mask<V>(w, k);
        acc.s += (double)slot_tree<V>(x);
    } else {
#pragma unroll
        for (int k = 0; k < V; ++k) acc.template add<OPC>(v[k], cell_mask<V>(w, k));
    }
}
template <class Acc, int OPC, int V, bool SM = false>
__device__ __forceinline__ void fold_full(Acc& acc, const uint32_t (&v)[V]) {
    if constexpr (tree_sum<Acc, OPC, V, SM>()) {
        acc.s += (double)slot_tree<V>(v);
    } else {
#pragma unroll
        for (int k = 0; k < V; ++k) acc.template add<OPC>(v[k], 0xFFFFFFFFu);
    }
}

// Byte-mask words of a run's first slot, last slot, and both (single-slot runs).
template <int V>
__device__ __forceinline__ void slot_masks(const QDesc& d, uint64_t& wf, uint64_t& wl, uint64_t& wb) {
    if (V == 1) {
        wf = wl = wb = ~0ull;
        return;
    }
    const int tail = (int)(d.h0 + d.L - (int64_t)V * (d.nslot - 1));  // cells of the last slot in the run
    const uint32_t full = (1u << V) - 1u;
    const uint32_t fm = full & ~((1u << d.h0) - 1u), lm = (1u << tail) - 1u;
    wf = byte_mask_word(fm);
    wl = byte_mask_word(lm);
    wb = byte_mask_word(fm & lm);
}

// loads in flight per lane: 32-B slots take 3 LDG.256 (long-run segments, and short runs of >= 16
// slots) or 2 (runs of < 16 slots, where a third mostly re-reads masked slots); 16-B / 4-B slots 4.
// Measured (profiles/sweep_r01_unroll.txt): C2a/C3/C4 gain 1-6% from the third load, C2b (runs of
// 1-5 slots) loses 20% with it.
#ifndef OLAP_U8
#define OLAP_U8 3
#endif
constexpr int unroll_for(int V) { return V == 8 ? OLAP_U8 : 4; }
#ifndef OLAP_SM_WIDE
#define OLAP_SM_WIDE 1  // tile path: wide mode for runs of > 32 slots (stream_wide)
#endif
#ifndef OLAP_SM_COLS
#define OLAP_SM_COLS 1  // tile path: column mode for runs of <= 32 slots (stream_cols)
#endif
#ifndef OLAP_SM_U
#define OLAP_SM_U 2  // tile path (shared-memory slots): slots in flight per lane
#endif

// Short runs (nslot <= kShortMaxSlots): a task is up to 31 whole runs.  Lane i holds
// the first-slot address of run r0+i.  The interior slots of all the task's runs
// (slots 1..nslot-2) are flattened and streamed WITHOUT masks: slot g is run
// j = g / (nslot-2) (fast division), slot 1 + g % (nslot-2), address via a shuffle.
// The two edge slots of every run go through a short masked pass.
template <class Acc, int OPC, int V, int U, bool SM = false>
__device__ __forceinline__ void stream_short(const uint32_t* __restrict__ cube, const QDesc& d, int64_t t0, int64_t t1,
                                             Acc& acc, int lane, int w, int ws) {
    int64_t t = t0 + w;
    if (t >= t1) return;
    const int rpt = d.T, nslot = (int)d.nslot;
    const int ni = nslot >= 2 ? nslot - 2 : 0, ne = nslot >= 2 ? 2 : 1;
    uint64_t wf, wl, wb;
    slot_masks<V>(d, wf, wl, wb);
    const FastDiv fni = d.fni;
    const int64_t R = d.R;
    for (; t < t1; t += ws) {
        const int64_t r0 = t * rpt;
        const int nr = (int)min((int64_t)rpt, R - r0);
        const int64_t ra = lane < nr ? run_addr(d, r0 + lane) : 0;
        const int nint = nr * ni;
        for (int i0 = 0; i0 < nint; i0 += 32 * U) {
            uint32_t v[U][V];
            bool ok[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int idx0 = i0 + 32 * u + lane;
                ok[u] = idx0 < nint;
                const int idx = ok[u] ? idx0 : nint - 1;  // re-read a valid slot, then drop it
                const int j = (int)fdiv((uint32_t)idx, fni);
                const int sl = 1 + idx - j * ni;
                load_slot<V, SM>(cube + __shfl_sync(0xffffffffu, ra, j & 31) + (int64_t)sl * V, v[u]);
            }
            if (i0 + 32 * U <= nint) {
#pragma unroll
                for (int u = 0; u < U; ++u) fold_full<Acc, OPC, V, SM>(acc, v[u]);
            } else {
#pragma unroll
                for (int u = 0; u < U; ++u) fold_slot<Acc, OPC, V, SM>(acc, v[u], ok[u] ? ~0ull : 0ull);
            }
        }
        const int nedge = nr * ne;
        for (int i0 = 0; i0 < nedge; i0 += 32 * U) {
            uint32_t v[U][V];
            uint64_t m[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int idx0 = i0 + 32 * u + lane;
                const bool ok = idx0 < nedge;
                const int idx = ok ? idx0 : nedge - 1;
                const int j = ne == 2 ? idx >> 1 : idx;
                const bool tailside = ne == 2 && (idx & 1);
                const int sl = tailside ? nslot - 1 : 0;
                m[u] = ok ? (nslot == 1 ? wb : (tailside ? wl : wf)) : 0ull;
                load_slot<V, SM>(cube + __shfl_sync(0xffffffffu, ra, j & 31) + (int64_t)sl * V, v[u]);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) fold_slot<Acc, OPC, V, SM>(acc, v[u], m[u]);
        }
    }
}

// Stream slots [0, count) of one run segment starting at slot address p (cells).
// wfirst / wlast: masks of slot 0 and slot count-1 (all ones when not a run edge;
// wboth when one slot is both).  Steps with no edge slot skip masking entirely.
template <class Acc, int OPC, int V, bool SM = false>
__device__ __forceinline__ void stream_segment(const uint32_t* __restrict__ p, int count, uint64_t wfirst,
                                               uint64_t wlast, uint64_t wboth, Acc& acc, int lane) {
    constexpr int U = unroll_for(V);
    for (int i0 = 0; i0 < count; i0 += 32 * U) {
        uint32_t v[U][V];
        uint64_t m[U];
        const bool interior = (i0 > 0 || wfirst == ~0ull) && (i0 + 32 * U < count || wlast == ~0ull) &&
                              i0 + 32 * U <= count;
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int idx0 = i0 + 32 * u + lane;
            const bool ok = idx0 < count;
            const int idx = ok ? idx0 : count - 1;  // re-read the last slot, masked out
            m[u] = ok ? (idx == 0 ? (idx == count - 1 ? wboth : wfirst) : (idx == count - 1 ? wlast : ~0ull)) : 0ull;
            load_slot<V, SM>(p + (int64_t)idx * V, v[u]);
        }
        if (interior) {
#pragma unroll
            for (int u = 0; u < U; ++u) fold_full<Acc, OPC, V, SM>(acc, v[u]);
        } else {
#pragma unroll
            for (int u = 0; u < U; ++u) fold_slot<Acc, OPC, V, SM>(acc, v[u], m[u]);
        }
    }
}

// Long runs (nslot > kShortMaxSlots): a task is kTaskSlots slots, at most two
// contiguous segments (the end of run j0 and the start of run j0+1).
template <class Acc, int OPC, int V, bool SM = false>
__device__ __forceinline__ void stream_long(const uint32_t* __restrict__ cube, const QDesc& d, int64_t t0, int64_t t1,
                                            Acc& acc, int lane, int w, int ws) {
    int64_t t = t0 + w;
    if (t >= t1) return;
    const int T_ = d.T;
    const int64_t nslot = d.nslot, G = d.G;
    uint64_t wf, wl, wb;
    slot_masks<V>(d, wf, wl, wb);
    int64_t j0 = div64(t * T_, nslot);
    int64_t rem = t * T_ - j0 * nslot;
    const int64_t step = (int64_t)ws * T_;
    for (; t < t1; t += ws) {
        const int64_t left = G - t * T_;
        const int n = left < T_ ? (int)left : T_;
        const int64_t in_run = nslot - rem;
        const int c1 = in_run < n ? (int)in_run : n;
        const bool first = rem == 0, lastin = rem + c1 == nslot;
        stream_segment<Acc, OPC, V, SM>(cube + run_addr(d, j0) + rem * V, c1, first ? wf : ~0ull, lastin ? wl : ~0ull,
                                    first && lastin ? wb : (first ? wf : wl), acc, lane);
        if (c1 < n) stream_segment<Acc, OPC, V, SM>(cube + run_addr(d, j0 + 1), n - c1, wf, ~0ull, wf, acc, lane);
        rem += step;
        if (rem >= nslot) {
            const int64_t dj = nslot < (1ll << 20) ? (int64_t)fdiv((uint32_t)rem, d.fnslot) : 1;
            j0 += dj;
            rem -= dj * nslot;
        }
    }
}

// Tasks t0+w, t0+w+ws, ... < t1 of one query's item (ws warps share the item).
// Tile path, runs of <= 32 slots whose start addresses need <= 2 digits (every pair of the
// benchmark cubes): "column mode".  Lane l owns slot s = l % nslot of run group l / nslot and
// keeps it for the whole pair, so its mask is fixed (built once) and the warp reads
// g = 32 / nslot whole runs per step, each as one contiguous span of shared memory (no
// per-slot division, no shuffle, no separate edge pass).  Idle lanes read lane 0's slot
// with an all-zero mask.  Offsets inside a staged tile fit in 32 bits.
// float MIN / MAX in column mode mask by addition on the FMA pipe instead of a LOP3 on the
// (binding) ALU pipe: m[k] holds a bias, +0.0 for a cell in the box and the op's identity
// (+inf for MIN, -inf for MAX) outside it, so v + bias is v or the identity (a NaN from
// -inf + inf is ignored by fminf / fmaxf; -0.0 + 0.0 reads as +0.0, reading R9).
template <class Acc, int OPC>
constexpr bool bias_fold() {
    return std::is_same<Acc, AccF>::value && (OPC == OPC_MIN || OPC == OPC_MAX);
}
template <int OPC>
constexpr uint32_t bias_identity() {
    return OPC == OPC_MIN ? 0x7f800000u : 0xff800000u;
}

template <class Acc, int OPC, int V>
__device__ __forceinline__ void fold_masked(Acc& acc, const uint32_t (&v)[V], const uint32_t (&m)[V]) {
    if constexpr (bias_fold<Acc, OPC>()) {
#pragma unroll
        for (int k = 0; k < V; ++k) {
            const float x = __uint_as_float(v[k]) + __uint_as_float(m[k]);
            if constexpr (OPC == OPC_MIN) acc.mn = fminf(acc.mn, x);
            else acc.mx = fmaxf(acc.mx, x);
        }
    } else if constexpr (tree_sum<Acc, OPC, V, true>()) {
        uint32_t x[V];
#pragma unroll
        for (int k = 0; k < V; ++k) x[k] = v[k] & m[k];
        acc.s += (double)slot_tree<V>(x);
    } else {
#pragma unroll
        for (int k = 0; k < V; ++k) acc.template add<OPC>(v[k], m[k]);
    }
}

__device__ __forceinline__ uint4 lds128(uint32_t a) {
    uint4 r;
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "r"(a));
    return r;
}
// one slot at shared byte addresses pa (cells 0-3 of v) and pb (cells 4-7; V == 8 only)
template <int V>
__device__ __forceinline__ void lds_slot(uint32_t pa, uint32_t pb, uint32_t (&v)[V]) {
    const uint4 x = lds128(pa);
    v[0] = x.x;
    v[1] = x.y;
    v[2] = x.z;
    v[3] = x.w;
    if constexpr (V == 8) {
        const uint4 y = lds128(pb);
        v[4] = y.x;
        v[5] = y.y;
        v[6] = y.z;
        v[7] = y.w;
    }
}

// NRD = digits of a run's start (0: one run; 1: r * rs0; 2: (r mod rad0) * rs0 + (r div rad0) * rs1).
// The lane's run advances by g per step; its offset is updated incrementally (one carry test).
// n / d for d in [1, 32] and n < 2^27 by one 64-bit multiply-high: q = (n * ceil(2^32 / d)) >> 32
// (exact: the excess n * (ceil(2^32/d) - 2^32/d) / 2^32 < 2^-5 <= 1/d); a runtime 32-bit division
// is ~20 instructions, and column mode needed three per pair
__constant__ unsigned long long kInv32[33] = {
    0ull,          4294967296ull, 2147483648ull, 1431655766ull, 1073741824ull, 858993460ull, 715827883ull,
    613566757ull,  536870912ull,  477218589ull,  429496730ull,  390451573ull,  357913942ull, 330382100ull,
    306783379ull,  286331154ull,  268435456ull,  252645136ull,  238609295ull,  226050911ull, 214748365ull,
    204522253ull,  195225787ull,  186737709ull,  178956971ull,  171798692ull,  165191050ull, 159072863ull,
    153391690ull,  148102321ull,  143165577ull,  138547333ull,  134217728ull};
__device__ __forceinline__ uint32_t div_le32(uint32_t n, uint32_t d) {
    return (uint32_t)(((unsigned long long)n * kInv32[d]) >> 32);
}

template <class Acc, int OPC, int V, int NRD>
__device__ __forceinline__ void stream_cols(const uint32_t* __restrict__ sb, const QDesc& d, Acc& acc, int lane) {
    static_assert(V == 4 || V == 8, "column mode reads 16-B slots");
    const uint32_t nslot = (uint32_t)d.nslot;
    const uint32_t g = div_le32(32u, nslot);  // nslot <= 32 in column mode
    const uint32_t grp = div_le32((uint32_t)lane, nslot);
    const uint32_t R = (uint32_t)d.R;
    const bool act = grp < g && grp < R;
    // idle lanes read the last active lane's slot (same address or the other half of it), so in a
    // partly idle quarter-warp they broadcast instead of bank-conflicting with the active lanes
    const uint32_t glast = (g < R ? g : R) - 1u;
    const uint32_t sl = act ? (uint32_t)lane - grp * nslot : nslot - 1u;
    uint64_t wf, wl, wb;
    slot_masks<V>(d, wf, wl, wb);
    uint64_t w = nslot == 1 ? wb : (sl == 0 ? wf : (sl == nslot - 1 ? wl : ~0ull));
    if (!act) w = 0;
    const bool swp = V == 8 && sm_swapped();
    if (swp) w = (w >> 32) | (w << 32);
    uint32_t m[V];
#pragma unroll
    for (int k = 0; k < V; ++k) {
        m[k] = cell_mask<V>(w, k);
        if constexpr (bias_fold<Acc, OPC>()) m[k] = ~m[k] & bias_identity<OPC>();
    }
    // lane byte addresses of its slot's two halves (half-swapped lanes read the upper half first)
    const uint32_t a0 = smem_addr_u32(sb) + ((uint32_t)d.base_al + sl * V) * 4u;
    const uint32_t pa = a0 + (swp ? 16u : 0u), pb = a0 + (swp ? 0u : 16u);
    const uint32_t my = act ? grp : glast;
    uint32_t off = 0, x0 = 0, rad0 = 1, s0 = 0, dstep = 0, dcarry = 0;
    if constexpr (NRD == 1) {
        const uint32_t rs0 = (uint32_t)d.rs[0] * 4u;
        off = my * rs0;
        dstep = g * rs0;
    } else if constexpr (NRD == 2) {
        const FastDiv f0 = d.frl[0];
        const uint32_t rs0 = (uint32_t)d.rs[0] * 4u, rs1 = (uint32_t)d.rs[1] * 4u;
        rad0 = f0.d;
        const uint32_t q = fdiv(my, f0), s1 = fdiv(g, f0);
        x0 = my - q * rad0;
        s0 = g - s1 * rad0;
        off = x0 * rs0 + q * rs1;
        dstep = s0 * rs0 + s1 * rs1;
        dcarry = rs1 - rad0 * rs0;
    }
    auto step = [&]() {
        off += dstep;
        if constexpr (NRD == 2) {
            x0 += s0;
            if (x0 >= rad0) {
                x0 -= rad0;
                off += dcarry;
            }
        }
    };
    const uint32_t full = div_le32(R, g) * g;  // steps in which every group has a run (R < 2^27: one tile / item)
    uint32_t r0 = 0;
    for (; r0 + 2 * g <= full; r0 += 2 * g) {
        uint32_t v0[V], v1[V];
        lds_slot<V>(pa + off, pb + off, v0);
        step();
        lds_slot<V>(pa + off, pb + off, v1);
        step();
        if constexpr (tree_sum<Acc, OPC, V, true>() && V == 8) {
            // float SUM: one fp32 tree over both slots (16 cells, depth 4; reading R8'), one fp64 add
            uint32_t x0[V], x1[V];
#pragma unroll
            for (int k = 0; k < V; ++k) {
                x0[k] = v0[k] & m[k];
                x1[k] = v1[k] & m[k];
            }
            acc.s += (double)(slot_tree<V>(x0) + slot_tree<V>(x1));
        } else {
            fold_masked<Acc, OPC, V>(acc, v0, m);
            fold_masked<Acc, OPC, V>(acc, v1, m);
        }
    }
    if (r0 < full) {
        uint32_t v0[V];
        lds_slot<V>(pa + off, pb + off, v0);
        step();
        fold_masked<Acc, OPC, V>(acc, v0, m);
        r0 += g;
    }
    if (r0 < R) {  // last, partial step: groups past the last run read run 0 and contribute identities
        const bool ok = r0 + my < R;
        const uint32_t okm = ok ? 0xFFFFFFFFu : 0u, o = ok ? off : 0u;
        uint32_t v0[V], mm[V];
        lds_slot<V>(pa + o, pb + o, v0);
#pragma unroll
        for (int k = 0; k < V; ++k) {
            if constexpr (bias_fold<Acc, OPC>()) mm[k] = m[k] | (~okm & bias_identity<OPC>());
            else mm[k] = m[k] & okm;
        }
        fold_masked<Acc, OPC, V>(acc, v0, mm);
    }
}

// Tile path, runs of > 32 slots (NRD as in stream_cols): "wide mode".  One run per step; lane l
// reads slots l, l+32, l+64, ... of it (32-slot chunks, 1 KiB apart: fixed offsets, no per-slot
// index arithmetic).  Only the first chunk (slot 0 in lane 0) and the last chunk (slot
// nslot-1, and lanes past the run end, which re-read the last slot with an all-zero mask)
// are masked; every chunk in between folds without masks.
template <class Acc, int OPC, int V, int NRD>
__device__ __forceinline__ void stream_wide(const uint32_t* __restrict__ sb, const QDesc& d, Acc& acc, int lane) {
    static_assert(V == 4 || V == 8, "wide mode reads 16-B slots");
    const uint32_t nslot = (uint32_t)d.nslot;
    const uint32_t K = (nslot + 31u) >> 5;  // chunks per run, >= 2
    const uint32_t R = (uint32_t)d.R;
    uint64_t wf, wl, wb;
    slot_masks<V>(d, wf, wl, wb);
    const uint32_t sl_last = (uint32_t)lane + 32u * (K - 1);
    const uint64_t w0 = lane == 0 ? wf : ~0ull;
    const uint64_t wL = sl_last == nslot - 1 ? wl : (sl_last < nslot ? ~0ull : 0ull);
    const bool swp = V == 8 && sm_swapped();
    const uint32_t a0 = smem_addr_u32(sb) + ((uint32_t)d.base_al + (uint32_t)lane * V) * 4u;
    const uint32_t pa = a0 + (swp ? 16u : 0u), pb = a0 + (swp ? 0u : 16u);
    constexpr uint32_t kChunk = 32u * V * 4u;  // bytes between a lane's consecutive slots
    const uint32_t lastoff = (min(sl_last, nslot - 1) - (uint32_t)lane) * V * 4u;
    uint32_t off = 0, x0 = 0, rad0 = 1, s1 = 0, rs0 = 0, rs1 = 0;
    if constexpr (NRD >= 1) rs0 = (uint32_t)d.rs[0] * 4u;
    if constexpr (NRD == 2) {
        rad0 = d.frl[0].d;
        rs1 = (uint32_t)d.rs[1] * 4u;
        s1 = rs1 - (rad0 - 1) * rs0;  // carry: x0 wraps to 0, next outer digit
    }
    for (uint32_t r = 0; r < R; ++r) {
        {
            uint32_t v0[V];
            lds_slot<V>(pa + off, pb + off, v0);
            fold_slot<Acc, OPC, V, true>(acc, v0, w0);
        }
        uint32_t k = 1;
        for (; k + 2 < K; k += 2) {
            uint32_t v0[V], v1[V];
            const uint32_t o0 = off + k * kChunk, o1 = o0 + kChunk;
            lds_slot<V>(pa + o0, pb + o0, v0);
            lds_slot<V>(pa + o1, pb + o1, v1);
            fold_full<Acc, OPC, V, true>(acc, v0);
            fold_full<Acc, OPC, V, true>(acc, v1);
        }
        if (k + 1 < K) {
            uint32_t v0[V];
            const uint32_t o0 = off + k * kChunk;
            lds_slot<V>(pa + o0, pb + o0, v0);
            fold_full<Acc, OPC, V, true>(acc, v0);
        }
        {
            uint32_t v0[V];
            lds_slot<V>(pa + off + lastoff, pb + off + lastoff, v0);
            fold_slot<Acc, OPC, V, true>(acc, v0, wL);
        }
        if constexpr (NRD == 1) {
            off += rs0;
        } else if constexpr (NRD == 2) {
            if (++x0 == rad0) {
                x0 = 0;
                off += s1;
            } else {
                off += rs0;
            }
        }
    }
}

template <typename T, class Acc, int OPC, int V, bool SM = false>
__device__ __forceinline__ void stream_tasks(const T* __restrict__ cube, const QDesc& d, int64_t t0, int64_t t1,
                                             Acc& acc, int lane, int w, int ws = kWarps) {
    const uint32_t* c = reinterpret_cast<const uint32_t*>(cube);
    if constexpr (SM && V >= 4) {
        if (OLAP_SM_COLS && d.shortp && d.nslot <= 32 && d.nrd <= 2) {
            if (d.nrd == 2) stream_cols<Acc, OPC, V, 2>(c, d, acc, lane);
            else if (d.nrd == 1) stream_cols<Acc, OPC, V, 1>(c, d, acc, lane);
            else stream_cols<Acc, OPC, V, 0>(c, d, acc, lane);
            return;
        }
        if (OLAP_SM_WIDE && d.nslot > 32 && d.nrd <= 2) {
            if (d.nrd == 2) stream_wide<Acc, OPC, V, 2>(c, d, acc, lane);
            else if (d.nrd == 1) stream_wide<Acc, OPC, V, 1>(c, d, acc, lane);
            else stream_wide<Acc, OPC, V, 0>(c, d, acc, lane);
            return;
        }
    }
    if (d.shortp) {
        if (SM) stream_short<Acc, OPC, V, OLAP_SM_U, SM>(c, d, t0, t1, acc, lane, w, ws);
        else if (V == 8 && d.nslot < 16) stream_short<Acc, OPC, V, 2, SM>(c, d, t0, t1, acc, lane, w, ws);
        else stream_short<Acc, OPC, V, unroll_for(V), SM>(c, d, t0, t1, acc, lane, w, ws);
    }
    else stream_long<Acc, OPC, V, SM>(c, d, t0, t1, acc, lane, w, ws);
}

// ------------------------------------------------------------------ plan

__device__ void build_desc(const Geo& g, const olap_range* r, int32_t op, QDesc& d) {
    d.opc = OPC_NONE;
    d.op = op;
    d.vlocal = 0;
    d.tasks = 0;
    d.G = 0;
    d.nrd = 0;
    d.tpi = 1;
    if (op < OLAP_SUM || op > OLAP_AVG) return;
    int64_t lo[kMaxDims], hi[kMaxDims];
    bool empty = false;
    for (int k = 0; k < g.nd; ++k) {
        lo[k] = r[k].lo;
        hi[k] = r[k].hi;
        if (lo[k] < 0 || hi[k] >= g.n[k]) return;  // invalid: flagged by finalize
        if (lo[k] > hi[k]) empty = true;
    }
    if (empty || op == OLAP_COUNT) return;  // COUNT = V needs no cell (Eq. 3, reading R5)
    int64_t llo, lhi;
    if (!shard_local_range(g.n[0], g.G, g.g, g.b, lo[0], hi[0], &llo, &lhi)) return;
    lo[0] = llo;
    hi[0] = lhi;
    int64_t ell[kMaxDims];
    for (int k = 0; k < g.nd; ++k) ell[k] = hi[k] - lo[k] + 1;
    int ks = g.nd - 1;  // split dim: innermost dim not fully covered (dims after it merge into runs)
    if (!g.padded)      // padding cells sit between innermost rows: such runs must not merge
        while (ks > 0 && ell[ks] == g.n[ks]) --ks;
    d.L = ell[ks] * g.stride[ks];
    int64_t R = 1, base = 0;
    for (int k = 0; k < g.nd; ++k) base += lo[k] * g.stride[k];
    int nrd = 0;
    bool a8 = true, a4 = true;
    for (int k = ks - 1; k >= 0; --k) {
        R *= ell[k];
        if (ell[k] > 1) {
            d.frl[nrd] = dev_fastdiv((uint32_t)ell[k]);
            d.rs[nrd] = g.stride[k];
            if (g.stride[k] & 7) a8 = false;
            if (g.stride[k] & 3) a4 = false;
            ++nrd;
        }
    }
    d.nrd = nrd;
    d.R = R;
    d.vlocal = R * d.L;
    // widest slot such that every run starts at the same offset inside its slot
    d.V = a8 ? 8 : (a4 ? 4 : 1);
    d.h0 = (int32_t)(base & (d.V - 1));
    d.base_al = base - d.h0;
    d.nslot = (d.h0 + d.L + d.V - 1) / d.V;
    d.G = R * d.nslot;
    if (d.nslot <= kShortMaxSlots) {  // short path: tasks of whole runs, <= 31 per task
        d.shortp = 1;
        int64_t rpt = kTaskSlots / d.nslot;
        rpt = rpt < 1 ? 1 : (rpt > 31 ? 31 : rpt);
        d.T = (int32_t)rpt;
        d.tasks = (R + rpt - 1) / rpt;
        d.fni = dev_fastdiv(d.nslot > 2 ? (uint32_t)(d.nslot - 2) : 1u);
        d.fnslot = dev_fastdiv(1u);
    } else {
        d.shortp = 0;
        d.T = d.nslot < kTaskSlots ? (int32_t)d.nslot : kTaskSlots;  // T <= nslot: a task spans <= 2 runs
        d.tasks = (d.G + d.T - 1) / d.T;
        d.fnslot = dev_fastdiv(d.nslot < (1ll << 31) ? (uint32_t)d.nslot : 1u);
        d.fni = dev_fastdiv(1u);
    }
    d.opc = (op == OLAP_MIN) ? OPC_MIN : (op == OLAP_MAX) ? OPC_MAX : OPC_SUM;
}

constexpr int kPlanThreads = 1024;

template <typename V>
__device__ V block_sum(V v, V* sh) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (lane == 0) sh[w] = v;
    __syncthreads();
    V t = 0;
    if (threadIdx.x < 32) {
        t = threadIdx.x < (blockDim.x >> 5) ? sh[threadIdx.x] : V(0);
#pragma unroll
        for (int o = 16; o; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
        if (threadIdx.x == 0) sh[0] = t;
    }
    __syncthreads();
    t = sh[0];
    __syncthreads();
    return t;
}

constexpr int kDescThreads = 256;

// Grid-wide, one thread per query: descriptor, identity partials for queries that read
// no cell, per-query (tasks, cells per task) for the scan, batch totals (atomics on
// integers: order-free, deterministic).
__global__ void __launch_bounds__(kDescThreads) desc_kernel(Geo geo, int64_t nq, const olap_range* __restrict__ ranges,
                                                            const int32_t* __restrict__ ops, QDesc* desc,
                                                            int64_t* q_tasks, int32_t* q_tv, int32_t* done,
                                                            int64_t* psum, int32_t* pext,
                                                            unsigned long long* totals, const int32_t* tmode) {
    if (*tmode) return;  // the tile-shared scan answers this batch
    __shared__ int64_t sh[32];
    const int64_t q = blockIdx.x * (int64_t)kDescThreads + threadIdx.x;
    int64_t cells = 0, slot_cells = 0;
    if (q < nq) {
        QDesc d;
        build_desc(geo, ranges + q * geo.nd, ops[q], d);
        desc[q] = d;
        done[q] = 0;
        if (d.opc == OPC_NONE) {
            psum[q] = 0;
            pext[2 * q] = INT_MIN;
            pext[2 * q + 1] = INT_MIN;
            q_tasks[q] = 0;
            q_tv[q] = 1;
        } else {
            cells = d.vlocal;
            slot_cells = d.G * d.V;
            q_tasks[q] = d.tasks;
            q_tv[q] = d.shortp ? (int32_t)(d.T * d.nslot * d.V) : d.T * d.V;  // cells per task
        }
    }
    cells = block_sum<int64_t>(cells, sh);
    slot_cells = block_sum<int64_t>(slot_cells, sh);
    if (threadIdx.x == 0) {
        if (cells) atomicAdd(totals + 0, (unsigned long long)cells);
        if (slot_cells) atomicAdd(totals + 1, (unsigned long long)slot_cells);
    }
}

// Item size (cells per item, "teff"): 1 MiB for block items, 256 KiB for warp items, smaller
// for small batches so that there are >= 4 items per worker (latency), and large enough that
// sum_q items_q <= items_cap: items_q <= tasks_q/tpi_q + 1 <= 2*G_q*V_q/teff + 2
// (tpi_q*T_q*V_q >= teff/2).
__device__ __forceinline__ int64_t item_cells(int64_t nq, int64_t items_cap, const unsigned long long* totals,
                                              int grid, int witems) {
    const int64_t total_slot_cells = (int64_t)totals[1];
    const int64_t cap_left = items_cap - 2 * nq;
    const int64_t workers = witems ? 8ll * grid : (int64_t)grid;
    const int64_t target = witems ? kItemCells / 4 : kItemCells;
    int64_t teff = total_slot_cells / (4ll * workers);
    if (teff > target) teff = target;
    const int64_t teff_cap = (4 * total_slot_cells + cap_left - 1) / cap_left;
    if (teff < teff_cap) teff = teff_cap;
    return teff < 1 ? 1 : teff;
}

// Items of query q (tasks-per-item written into its descriptor).
__device__ __forceinline__ int64_t query_items(QDesc* desc, const int64_t* __restrict__ q_tasks,
                                               const int32_t* __restrict__ q_tv, int64_t q, int64_t teff) {
    const int64_t tasks = q_tasks[q];
    if (!tasks) return 0;
    int64_t tpi = teff / q_tv[q];
    if (tpi < 1) tpi = 1;
    if (tpi > (1ll << 30)) tpi = (1ll << 30);
    desc[q].tpi = (int32_t)tpi;
    return (tasks + tpi - 1) / tpi;
}

// Grid-wide, one thread per query: item count per query (icnt[nq] = 0); a CUB exclusive
// scan then gives item_start[0..nq].  Large batches (> kPlanSmall queries).
__global__ void items_kernel(int64_t nq, QDesc* desc, const int64_t* __restrict__ q_tasks,
                             const int32_t* __restrict__ q_tv, int64_t* __restrict__ icnt, int64_t items_cap,
                             const unsigned long long* totals, int grid, int witems, const int32_t* tmode) {
    if (*tmode) return;
    const int64_t teff = item_cells(nq, items_cap, totals, grid, witems);
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q <= nq; q += (int64_t)gridDim.x * blockDim.x)
        icnt[q] = q < nq ? query_items(desc, q_tasks, q_tv, q, teff) : 0;
}

// Small batches (<= kPlanSmall queries): items, exclusive scan and the scan_fix_kernel work
// in one block (one launch instead of four; C1's 1,000-query batches are launch-bound).
constexpr int64_t kPlanSmall = 16384;
__global__ void __launch_bounds__(kPlanThreads) plan_small_kernel(int64_t nq, QDesc* desc,
                                                                  const int64_t* __restrict__ q_tasks,
                                                                  const int32_t* __restrict__ q_tv,
                                                                  int64_t* __restrict__ item_start,
                                                                  unsigned long long* counter, int64_t items_cap,
                                                                  const unsigned long long* totals,
                                                                  unsigned long long* bytes_acc, int grid, int witems,
                                                                  const int32_t* tmode) {
    if (*tmode) return;
    const int tid = threadIdx.x;
    const int64_t teff = item_cells(nq, items_cap, totals, grid, witems);
    const int64_t per = (nq + kPlanThreads - 1) / kPlanThreads;
    const int64_t q0 = min(nq, (int64_t)tid * per), q1 = min(nq, q0 + per);
    int64_t mine = 0;
    for (int64_t q = q0; q < q1; ++q) {
        const int64_t it = query_items(desc, q_tasks, q_tv, q, teff);
        item_start[q] = it;
        mine += it;
    }
    __shared__ int64_t scan[kPlanThreads];
    scan[tid] = mine;
    __syncthreads();
    for (int o = 1; o < kPlanThreads; o <<= 1) {
        const int64_t v = tid >= o ? scan[tid - o] : 0;
        __syncthreads();
        scan[tid] += v;
        __syncthreads();
    }
    int64_t off = scan[tid] - mine;
    for (int64_t q = q0; q < q1; ++q) {
        const int64_t it = item_start[q];
        item_start[q] = off;
        off += it;
    }
    if (tid == kPlanThreads - 1) {
        if (scan[tid] > items_cap) __trap();  // impossible by item_cells' bound
        item_start[nq] = scan[tid];
        *counter = 0ull;
        atomicAdd(bytes_acc, (unsigned long long)(totals[0] * 4));
    }
}

// After the scan: bound check, reset the item counter, count the batch's algorithmic bytes.
__global__ void scan_fix_kernel(int64_t nq, const int64_t* __restrict__ item_start, unsigned long long* counter,
                                int64_t items_cap, const unsigned long long* totals, unsigned long long* bytes_acc,
                                const int32_t* tmode) {
    if (tmode && *tmode) return;
    // never write past the item-partial arrays: fail loudly instead (cannot happen by the bound above)
    if (item_start[nq] > items_cap) __trap();
    *counter = 0ull;
    atomicAdd(bytes_acc, (unsigned long long)(totals[0] * 4));
}

// ------------------------------------------------------------------ L2-aware item order
// Items are popped in order of the cube address they start at (counting sort into
// buckets of bucket_cells), so the ~600 blocks resident at any moment work on the same
// few MiB of the cube and the many queries that cover it (C2a: ~400x per batch) hit
// in the 126 MB L2 instead of re-reading HBM.  Partials stay indexed by item id and are
// folded in fixed order, so results do not depend on this order.
constexpr int kMaxBuckets = 4096;

__device__ __forceinline__ int64_t find_query_thread(const int64_t* __restrict__ item_start, int64_t nq,
                                                     int64_t item) {
    int64_t lo = 0, hi = nq;  // largest q with item_start[q] <= item
    while (hi - lo > 1) {
        const int64_t mid = (lo + hi) >> 1;
        if (__ldg(item_start + mid) <= item) lo = mid;
        else hi = mid;
    }
    return lo;
}

__global__ void bucket_kernel(int64_t nq, const QDesc* __restrict__ desc, const int64_t* __restrict__ item_start,
                              int shift, int32_t* __restrict__ bucket, unsigned int* count, const int32_t* tmode) {
    if (*tmode) return;
    const int64_t total = __ldg(item_start + nq);
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t q = find_query_thread(item_start, nq, i);
        const QDesc& d = desc[q];
        const int64_t t0 = (i - __ldg(item_start + q)) * (int64_t)d.tpi;  // first task of the item
        int64_t addr;
        if (d.shortp) {
            addr = run_addr(d, t0 * d.T);
        } else {
            const int64_t g = t0 * d.T, j = g / d.nslot;
            addr = run_addr(d, j) + (g - j * d.nslot) * d.V;
        }
        int64_t b = addr >> shift;
        if (b >= kMaxBuckets) b = kMaxBuckets - 1;
        bucket[i] = (int32_t)b;
        atomicAdd(count + b, 1u);
    }
}

__global__ void __launch_bounds__(1024) bucket_scan_kernel(unsigned int* count, unsigned int* cursor,
                                                           const int32_t* tmode) {
    if (*tmode) return;
    __shared__ unsigned int sh[kMaxBuckets];
    for (int b = threadIdx.x; b < kMaxBuckets; b += blockDim.x) sh[b] = count[b];
    __syncthreads();
    if (threadIdx.x == 0) {  // 4096 entries: a serial scan is ~10 us and simplest
        unsigned int acc = 0;
        for (int b = 0; b < kMaxBuckets; ++b) {
            const unsigned int c = sh[b];
            sh[b] = acc;
            acc += c;
        }
    }
    __syncthreads();
    for (int b = threadIdx.x; b < kMaxBuckets; b += blockDim.x) cursor[b] = sh[b];
}

__global__ void scatter_kernel(int64_t nq, const int64_t* __restrict__ item_start, const int32_t* __restrict__ bucket,
                               unsigned int* cursor, int32_t* __restrict__ order, const int32_t* tmode) {
    if (*tmode) return;
    const int64_t total = __ldg(item_start + nq);
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x)
        order[atomicAdd(cursor + bucket[i], 1u)] = (int32_t)i;
}

// ------------------------------------------------------------------ reduce (the hot loop)

// op-class x slot-width dispatch of one item's tasks
template <typename T, class Acc, bool SM = false>
__device__ __forceinline__ void stream_item(const T* __restrict__ cube, const QDesc& sd, int64_t t0, int64_t t1, Acc& acc,
                                            int lane, int w, int ws) {
    const int opc = sd.opc;
    if (sd.V == 8) {
        if (opc == OPC_SUM) stream_tasks<T, Acc, OPC_SUM, 8, SM>(cube, sd, t0, t1, acc, lane, w, ws);
        else if (opc == OPC_MIN) stream_tasks<T, Acc, OPC_MIN, 8, SM>(cube, sd, t0, t1, acc, lane, w, ws);
        else stream_tasks<T, Acc, OPC_MAX, 8, SM>(cube, sd, t0, t1, acc, lane, w, ws);
    } else if (sd.V == 4) {
        if (opc == OPC_SUM) stream_tasks<T, Acc, OPC_SUM, 4, SM>(cube, sd, t0, t1, acc, lane, w, ws);
        else if (opc == OPC_MIN) stream_tasks<T, Acc, OPC_MIN, 4, SM>(cube, sd, t0, t1, acc, lane, w, ws);
        else stream_tasks<T, Acc, OPC_MAX, 4, SM>(cube, sd, t0, t1, acc, lane, w, ws);
    } else if constexpr (!SM) {  // tile path: every run stride is a multiple of 4 cells (V >= 4)
        if (opc == OPC_SUM) stream_tasks<T, Acc, OPC_SUM, 1, SM>(cube, sd, t0, t1, acc, lane, w, ws);
        else if (opc == OPC_MIN) stream_tasks<T, Acc, OPC_MIN, 1, SM>(cube, sd, t0, t1, acc, lane, w, ws);
        else stream_tasks<T, Acc, OPC_MAX, 1, SM>(cube, sd, t0, t1, acc, lane, w, ws);
    }
}

// Warp-granular variant: every warp pops its own item, streams all of its tasks, and the
// last warp to finish a query folds its item partials — no block barriers at all.
template <typename T, class Acc>
__global__ void __launch_bounds__(kThreads, kMinBlocks) reduce_kernel_w(const T* __restrict__ cube, int64_t nq,
                                                               const QDesc* __restrict__ desc,
                                                               const int64_t* __restrict__ item_start,
                                                               unsigned long long* counter, int32_t* done,
                                                               long long* item_sum, int32_t* item_ext, int64_t* psum,
                                                               int32_t* pext, const int32_t* __restrict__ order,
                                                               const int32_t* tmode) {
    if (*tmode) return;
    __shared__ QDesc sdw[kWarps];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    QDesc& sd = sdw[w];
    const int64_t total = __ldg(item_start + nq);
    for (;;) {
        long long item = 0;
        if (lane == 0) {
            const int64_t slot = (int64_t)atomicAdd(counter, 1ull);
            item = (order && slot < total) ? (long long)__ldg(order + slot) : (long long)slot;
        }
        item = __shfl_sync(0xffffffffu, item, 0);
        if (item >= total) break;
        const int64_t q = find_query(item_start, nq, item, lane);
        {
            const int* src = reinterpret_cast<const int*>(desc + q);
            int* dst = reinterpret_cast<int*>(&sd);
            for (int i = lane; i < (int)(sizeof(QDesc) / 4); i += 32) dst[i] = __ldg(src + i);
        }
        __syncwarp();
        const int64_t first_item = __ldg(item_start + q);
        const int64_t t0 = (item - first_item) * (int64_t)sd.tpi;
        const int64_t t1 = min(sd.tasks, t0 + (int64_t)sd.tpi);
        Acc acc;
        acc.init();
        const int opc = sd.opc;
        stream_item<T, Acc>(cube, sd, t0, t1, acc, lane, 0, 1);
        long long s = acc.sum_bits();
        int32_t cmx = opc == OPC_MAX ? acc.code_max() : INT_MIN, cmn = opc == OPC_MIN ? ~acc.code_min() : INT_MIN;
#pragma unroll
        for (int o = 16; o; o >>= 1) s = SumOps<Acc>::add(s, __shfl_xor_sync(0xffffffffu, s, o));
        cmx = __reduce_max_sync(0xffffffffu, cmx);
        cmn = __reduce_max_sync(0xffffffffu, cmn);
        const int64_t nitems = (sd.tasks + sd.tpi - 1) / sd.tpi;
        int last = 0;
        if (lane == 0) {
            item_sum[item] = s;
            item_ext[2 * item] = cmx;
            item_ext[2 * item + 1] = cmn;
            __threadfence();
            last = atomicAdd(done + q, 1) == (int)nitems - 1;
        }
        last = __shfl_sync(0xffffffffu, last, 0);
        if (last) {  // fold the query's item partials in fixed order
            __threadfence();
            long long ts = 0;
            int32_t tmx = INT_MIN, tmn = INT_MIN;
            for (int64_t i = lane; i < nitems; i += 32) {
                const int64_t it = first_item + i;
                ts = SumOps<Acc>::add(ts, __ldcg(item_sum + it));
                tmx = max(tmx, __ldcg(item_ext + 2 * it));
                tmn = max(tmn, __ldcg(item_ext + 2 * it + 1));
            }
#pragma unroll
            for (int o = 16; o; o >>= 1) ts = SumOps<Acc>::add(ts, __shfl_xor_sync(0xffffffffu, ts, o));
            tmx = __reduce_max_sync(0xffffffffu, tmx);
            tmn = __reduce_max_sync(0xffffffffu, tmn);
            if (lane == 0) {
                psum[q] = ts;
                pext[2 * q] = tmx;
                pext[2 * q + 1] = tmn;
            }
        }
        __syncwarp();
    }
}

template <typename T, class Acc>
__global__ void __launch_bounds__(kThreads, kMinBlocks) reduce_kernel(const T* __restrict__ cube, int64_t nq,
                                                             const QDesc* __restrict__ desc,
                                                             const int64_t* __restrict__ item_start,
                                                             unsigned long long* counter, int32_t* done,
                                                             long long* item_sum, int32_t* item_ext, int64_t* psum,
                                                             int32_t* pext, const int32_t* __restrict__ order,
                                                             const int32_t* tmode) {
    if (*tmode) return;
    __shared__ QDesc sd;
    __shared__ int64_t s_item, s_q;
    __shared__ long long s_wsum[kWarps];
    __shared__ int32_t s_wmx[kWarps], s_wmn[kWarps];
    __shared__ int s_last;

    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t total = __ldg(item_start + nq);

    for (;;) {
        if (threadIdx.x == 0) {
            const int64_t slot = (int64_t)atomicAdd(counter, 1ull);
            s_item = (order && slot < total) ? (int64_t)__ldg(order + slot) : slot;
        }
        __syncthreads();
        const int64_t item = s_item;
        if (item >= total) break;
        if (w == 0) {
            const int64_t q = find_query(item_start, nq, item, lane);
            if (lane == 0) s_q = q;
        }
        __syncthreads();
        const int64_t q = s_q;
        {
            const int* src = reinterpret_cast<const int*>(desc + q);
            int* dst = reinterpret_cast<int*>(&sd);
            for (int i = threadIdx.x; i < (int)(sizeof(QDesc) / 4); i += kThreads) dst[i] = __ldg(src + i);
        }
        __syncthreads();
        const int64_t first_item = __ldg(item_start + q);
        const int64_t t0 = (item - first_item) * (int64_t)sd.tpi;
        const int64_t t1 = min(sd.tasks, t0 + (int64_t)sd.tpi);

        Acc acc;
        acc.init();
        const int opc = sd.opc;
        stream_item<T, Acc>(cube, sd, t0, t1, acc, lane, w, kWarps);

        // warp -> block -> item partial (fixed order: deterministic)
        long long s = acc.sum_bits();
        int32_t cmx = acc.code_max(), cmn = ~acc.code_min();
        if (opc != OPC_MAX) cmx = INT_MIN;
        if (opc != OPC_MIN) cmn = INT_MIN;
#pragma unroll
        for (int o = 16; o; o >>= 1) s = SumOps<Acc>::add(s, __shfl_xor_sync(0xffffffffu, s, o));
        cmx = __reduce_max_sync(0xffffffffu, cmx);
        cmn = __reduce_max_sync(0xffffffffu, cmn);
        if (lane == 0) {
            s_wsum[w] = s;
            s_wmx[w] = cmx;
            s_wmn[w] = cmn;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            long long ts = s_wsum[0];
            int32_t tmx = s_wmx[0], tmn = s_wmn[0];
#pragma unroll
            for (int i = 1; i < kWarps; ++i) {
                ts = SumOps<Acc>::add(ts, s_wsum[i]);
                tmx = max(tmx, s_wmx[i]);
                tmn = max(tmn, s_wmn[i]);
            }
            item_sum[item] = ts;
            item_ext[2 * item] = tmx;
            item_ext[2 * item + 1] = tmn;
            __threadfence();
            const int64_t nitems = (sd.tasks + sd.tpi - 1) / sd.tpi;
            const int prev = atomicAdd(done + q, 1);
            s_last = (prev == (int)nitems - 1);
        }
        __syncthreads();
        if (s_last) {
            // last finisher of query q: fold its item partials in fixed order
            __threadfence();
            const int64_t nitems = (sd.tasks + sd.tpi - 1) / sd.tpi;
            long long ts = 0;
            int32_t tmx = INT_MIN, tmn = INT_MIN;
            for (int64_t i = threadIdx.x; i < nitems; i += kThreads) {
                const int64_t it = first_item + i;
                ts = SumOps<Acc>::add(ts, __ldcg(item_sum + it));
                tmx = max(tmx, __ldcg(item_ext + 2 * it));
                tmn = max(tmn, __ldcg(item_ext + 2 * it + 1));
            }
#pragma unroll
            for (int o = 16; o; o >>= 1) ts = SumOps<Acc>::add(ts, __shfl_xor_sync(0xffffffffu, ts, o));
            tmx = __reduce_max_sync(0xffffffffu, tmx);
            tmn = __reduce_max_sync(0xffffffffu, tmn);
            if (lane == 0) {
                s_wsum[w] = ts;
                s_wmx[w] = tmx;
                s_wmn[w] = tmn;
            }
            __syncthreads();
            if (threadIdx.x == 0) {
                long long fs = s_wsum[0];
                int32_t fmx = s_wmx[0], fmn = s_wmn[0];
#pragma unroll
                for (int i = 1; i < kWarps; ++i) {
                    fs = SumOps<Acc>::add(fs, s_wsum[i]);
                    fmx = max(fmx, s_wmx[i]);
                    fmn = max(fmn, s_wmn[i]);
                }
                psum[q] = fs;
                pext[2 * q] = fmx;
                pext[2 * q + 1] = fmn;
            }
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------------ bricked cubes: brick_reduce_kernel
// A query on a bricked cube (OLAP_LAYOUT_BRICK / OLAP_LAYOUT_BRICK3; the layouts themselves are
// defined below, before the host runtime) is its box of bricks: the leading dims' ranges x the
// bricks [W0, W1] x [X0, X1] x [Z0, Z1] its x_{N-3} / x_{N-2} / x_{N-1} ranges meet.  A lane quad
// takes one 128-B brick per step (one LDG.256 per lane, all in flight), masks the cells outside
// the box (only in the box's edge bricks) and folds its 8 cells: one DRAM fetch line per brick
// (reading R26).  Brick shapes (cells along x_{N-3}, x_{N-2}, x_{N-1}):
//   BS = 0: 1 x 4 x 8 (OLAP_LAYOUT_BRICK), BS = 1: 2 x 4 x 4 (OLAP_LAYOUT_BRICK3).
template <int BS> struct BrickShape;
template <> struct BrickShape<0> { static constexpr int A0 = 1, A = 4, B = 8; };
template <> struct BrickShape<1> { static constexpr int A0 = 2, A = 4, B = 4; };
constexpr int kBrickDims = kMaxDims - 3;  // leading dims 0..N-4 (N <= kMaxDims - 2)
struct BDesc {
    int32_t opc, nld;          // op class; leading digits (dims 0..N-4 with extent > 1)
    int32_t wa, wb, ya, yb, za, zb;  // first brick's first / last brick's last cell along x_{N-3}, x_{N-2}, x_{N-1}
    int64_t nb;                // bricks in the box (0: reads nothing)
    int64_t base;              // cell offset of the box's first brick
    int64_t sW, sX;            // cells between bricks along x_{N-3}, x_{N-2} (Z stride is 32)
    FastDiv fZ, fX, fW;        // / nZ, / nX, / nW (brick extents of the box)
    FastDiv fl[kBrickDims];    // / leading extents, innermost first (the outermost is not divided)
    int64_t sl[kBrickDims];    // leading strides (cells), innermost first
};
static_assert(sizeof(BDesc) <= sizeof(QDesc), "brick descriptors live in the QDesc workspace");

// Geometry of the brick array of a bricked cube (shard-local).
struct BGeo {
    int nd;                    // logical dims N
    int64_t G, g, b;           // dim-0 shards
    int64_t n[kMaxDims];       // logical global extents
    int64_t stride[kMaxDims];  // brick-array strides (cells) of dims 0..N-4, then W (N-3), X (N-2); Z stride is 32
    int64_t local_rows;
};

// One thread per query: the box of bricks on this shard, identity partials when it reads
// nothing, per-query brick counts for the item planner, batch totals (cells, bricks).
template <int BS>
__global__ void __launch_bounds__(256) brick_desc_kernel(BGeo g, int64_t nq, const olap_range* __restrict__ ranges,
                                                         const int32_t* __restrict__ ops, BDesc* __restrict__ desc,
                                                         int64_t* __restrict__ q_bricks, int32_t* __restrict__ done,
                                                         int64_t* __restrict__ psum, int32_t* __restrict__ pext,
                                                         unsigned long long* totals) {
    using S = BrickShape<BS>;
    __shared__ int64_t sh[32];
    const int64_t q = blockIdx.x * 256ll + threadIdx.x;
    int64_t cells = 0, bricks = 0;
    if (q < nq) {
        const olap_range* r = ranges + q * g.nd;
        const int32_t op = ops[q];
        BDesc d;
        d.nb = 0;
        d.opc = (op == OLAP_MIN) ? OPC_MIN : (op == OLAP_MAX) ? OPC_MAX : OPC_SUM;
        bool ok = op == OLAP_SUM || op == OLAP_MIN || op == OLAP_MAX || op == OLAP_AVG;
        for (int k = 0; k < g.nd; ++k) ok = ok && r[k].lo >= 0 && r[k].hi < g.n[k] && r[k].lo <= r[k].hi;
        int64_t l0 = 0, h0 = -1;
        if (ok) ok = shard_local_range(g.n[0], g.G, g.g, g.b, r[0].lo, r[0].hi, &l0, &h0);
        if (ok) {
            const int wd = g.nd - 3, a = g.nd - 2, bz = g.nd - 1;
            // x_{N-3} in shard-local coordinates (dim 0 when N = 3: the owned rows are one local range)
            const int64_t wlo = wd == 0 ? l0 : r[wd].lo, whi = wd == 0 ? h0 : r[wd].hi;
            const int64_t W0 = wlo / S::A0, W1 = whi / S::A0;
            const int64_t X0 = r[a].lo / S::A, X1 = r[a].hi / S::A, Z0 = r[bz].lo / S::B, Z1 = r[bz].hi / S::B;
            d.wa = (int32_t)(wlo % S::A0);
            d.wb = (int32_t)(whi % S::A0);
            d.ya = (int32_t)(r[a].lo % S::A);
            d.yb = (int32_t)(r[a].hi % S::A);
            d.za = (int32_t)(r[bz].lo % S::B);
            d.zb = (int32_t)(r[bz].hi % S::B);
            const int64_t nW = W1 - W0 + 1, nX = X1 - X0 + 1, nZ = Z1 - Z0 + 1;
            d.sW = g.stride[wd];
            d.sX = g.stride[a];
            d.fW = dev_fastdiv((uint32_t)nW);
            d.fX = dev_fastdiv((uint32_t)nX);
            d.fZ = dev_fastdiv((uint32_t)nZ);
            int64_t base = W0 * d.sW + X0 * d.sX + Z0 * 32, nb = nW * nX * nZ;
            int64_t v = (whi - wlo + 1) * (r[a].hi - r[a].lo + 1) * (r[bz].hi - r[bz].lo + 1);
            int nld = 0;
            for (int k = wd - 1; k >= 0; --k) {
                const int64_t lo = k == 0 ? l0 : r[k].lo, hi = k == 0 ? h0 : r[k].hi, ell = hi - lo + 1;
                base += lo * g.stride[k];
                nb *= ell;
                v *= ell;
                if (ell > 1) {
                    d.fl[nld] = dev_fastdiv((uint32_t)ell);
                    d.sl[nld] = g.stride[k];
                    ++nld;
                }
            }
            d.nld = nld;
            d.base = base;
            d.nb = nb;
            cells = v;
            bricks = nb;
        }
        desc[q] = d;
        done[q] = 0;
        q_bricks[q] = d.nb;
        if (d.nb == 0 || op == OLAP_COUNT) {
            if (op == OLAP_COUNT) q_bricks[q] = 0, cells = 0, bricks = 0;
            psum[q] = 0;
            pext[2 * q] = INT_MIN;
            pext[2 * q + 1] = INT_MIN;
        }
    }
    cells = block_sum<int64_t>(cells, sh);
    bricks = block_sum<int64_t>(bricks, sh);
    if (threadIdx.x == 0) {
        if (cells) atomicAdd(totals + 0, (unsigned long long)cells);
        if (bricks) atomicAdd(totals + 1, (unsigned long long)bricks);
    }
}

// Bricks per item: <= 1,024 (32 warp steps of 32 bricks), fewer for small batches (>= 4 items per warp
// slot), more if the item-partial arrays would overflow (items_q <= bricks_q / bpi + 1).
__global__ void brick_items_kernel(int64_t nq, BDesc* desc, const int64_t* __restrict__ q_bricks,
                                   int64_t* __restrict__ icnt, int64_t items_cap, const unsigned long long* totals,
                                   int warps) {
    const int64_t total = (int64_t)totals[1];
    int64_t bpi = total / (4ll * warps);
    if (bpi > 1024) bpi = 1024;
    const int64_t cap_left = items_cap - nq;
    const int64_t bpi_cap = (total + cap_left - 1) / cap_left;
    if (bpi < bpi_cap) bpi = bpi_cap;
    if (bpi < 32) bpi = 32;
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q <= nq; q += (int64_t)gridDim.x * blockDim.x) {
        const int64_t nb = q < nq ? q_bricks[q] : 0;
        icnt[q] = (nb + bpi - 1) / bpi;
        if (q == 0) icnt[nq + 1] = bpi;  // read by brick_reduce_kernel (icnt has nq + 2 entries)
    }
}

__device__ __forceinline__ uint64_t byte_range_word(int lo, int hi) {  // bytes lo..hi of 8 = 0xFF
    return (~0ull << (8 * lo)) & (~0ull >> (8 * (7 - hi)));
}

// Cell offset of brick j (< 2^32) of the box: Z fastest, then X, then W, then the leading digits.
__device__ __forceinline__ int64_t brick_addr(const BDesc& d, uint32_t j, uint32_t& W, uint32_t& X, uint32_t& Z) {
    uint32_t t = fdiv(j, d.fZ);
    Z = j - t * d.fZ.d;
    const uint32_t t2 = fdiv(t, d.fX);
    X = t - t2 * d.fX.d;
    t = t2;
    if (d.nld == 0) {  // W is the outermost digit: no division
        W = t;
        return d.base + (int64_t)Z * 32 + (int64_t)X * d.sX + (int64_t)W * d.sW;
    }
    const uint32_t t3 = fdiv(t, d.fW);
    W = t - t3 * d.fW.d;
    int64_t a = d.base + (int64_t)Z * 32 + (int64_t)X * d.sX + (int64_t)W * d.sW;
    t = t3;
    for (int e = 0; e < d.nld; ++e) {
        if (e == d.nld - 1) {  // outermost digit: no division
            a += (int64_t)t * d.sl[e];
            break;
        }
        const uint32_t qq = fdiv(t, d.fl[e]);
        a += (int64_t)(t - qq * d.fl[e].d) * d.sl[e];
        t = qq;
    }
    return a;
}

template <class Acc, int OPC>
__device__ __forceinline__ void fold_row(Acc& acc, const uint32_t (&v)[8], uint64_t w) {
    if constexpr (OPC == OPC_SUM && std::is_same<Acc, AccF>::value) {  // fp32 tree of 8 cells (R8'), then fp64
        uint32_t x[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) x[k] = v[k] & cell_mask<8>(w, k);
        acc.s += (double)slot_tree<8>(x);
    } else {
#pragma unroll
        for (int k = 0; k < 8; ++k) acc.template add<OPC>(v[k], cell_mask<8>(w, k));
    }
}

// Byte mask of the 8 cells lane quad member `y4` holds in brick (W, X, Z) (cells 8 y4 .. 8 y4 + 7 of
// the brick, stored (w, y, z) with z fastest).
template <int BS>
__device__ __forceinline__ uint64_t brick_quad_mask(const BDesc& d, int y4, uint32_t W, uint32_t X, uint32_t Z) {
    using S = BrickShape<BS>;
    const int ylo = X == 0 ? d.ya : 0, yhi = X == d.fX.d - 1 ? d.yb : S::A - 1;
    const int zlo = Z == 0 ? d.za : 0, zhi = Z == d.fZ.d - 1 ? d.zb : S::B - 1;
    if constexpr (BS == 0) {  // the quad member is brick row y = y4: 8 cells along z
        return y4 >= ylo && y4 <= yhi ? byte_range_word(zlo, zhi) : 0ull;
    } else {  // w = y4 / 2; rows y = 2 (y4 & 1) and +1, 4 cells along z each
        const int w = y4 >> 1, wlo = W == 0 ? d.wa : 0, whi = W == d.fW.d - 1 ? d.wb : S::A0 - 1;
        if (w < wlo || w > whi) return 0ull;
        const uint32_t zm = (uint32_t)byte_range_word(zlo, zhi);  // bytes zlo..zhi of 4
        const int y = 2 * (y4 & 1);
        return (y >= ylo && y <= yhi ? (uint64_t)zm : 0ull) | (y + 1 >= ylo && y + 1 <= yhi ? (uint64_t)zm << 32 : 0ull);
    }
}

// Four lanes per brick (lane quad = one 128-B line, one coalesced request), 8 bricks per warp
// step, kBrickU steps of loads in flight per lane.
#ifndef OLAP_BRICK_U
#define OLAP_BRICK_U 3
#endif
constexpr int kBrickU = OLAP_BRICK_U;
template <class Acc, int OPC, int BS>
__device__ __forceinline__ void stream_bricks(const uint32_t* __restrict__ cube, const BDesc& d, int64_t b0,
                                              int64_t b1, Acc& acc, int lane) {
    const int sub = lane >> 2, y4 = lane & 3;
    for (int64_t j0 = b0; j0 < b1; j0 += 8 * kBrickU) {
        uint32_t v[kBrickU][8];
        uint64_t w[kBrickU];
#pragma unroll
        for (int u = 0; u < kBrickU; ++u) {
            const int64_t j = j0 + 8 * u + sub;
            const bool ok = j < b1;
            const int64_t jj = ok ? j : b1 - 1;  // < 2^32: a shard holds < 2^32 bricks (checked at creation)
            uint32_t W, X, Z;
            const int64_t a = brick_addr(d, (uint32_t)jj, W, X, Z);
            ld_stream8(cube + a + 8 * y4, v[u]);
            w[u] = ok ? brick_quad_mask<BS>(d, y4, W, X, Z) : 0ull;
        }
#pragma unroll
        for (int u = 0; u < kBrickU; ++u) fold_row<Acc, OPC>(acc, v[u], w[u]);
    }
}

// Persistent warp-item kernel over (query, brick range) items; partials folded per query in
// fixed item order by the query's last warp (as reduce_kernel_w: deterministic).
#ifndef OLAP_BRICK_BLOCKS
#define OLAP_BRICK_BLOCKS 3
#endif
constexpr int kBrickBlocks = OLAP_BRICK_BLOCKS;  // resident blocks per SM the register budget targets
template <typename T, class Acc, int BS>
__global__ void __launch_bounds__(kThreads, kBrickBlocks) brick_reduce_kernel(
    const T* __restrict__ cube, int64_t nq, const BDesc* __restrict__ desc, const int64_t* __restrict__ item_start,
    const int64_t* __restrict__ icnt, unsigned long long* counter, int32_t* done, long long* item_sum,
    int32_t* item_ext, int64_t* psum, int32_t* pext) {
    __shared__ BDesc sdw[kWarps];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    BDesc& sd = sdw[w];
    const int64_t total = __ldg(item_start + nq), bpi = __ldg(icnt + nq + 1);
    const uint32_t* c = reinterpret_cast<const uint32_t*>(cube);
    for (;;) {
        long long item = 0;
        if (lane == 0) item = (long long)atomicAdd(counter, 1ull);
        item = __shfl_sync(0xffffffffu, item, 0);
        if (item >= total) break;
        const int64_t q = find_query(item_start, nq, item, lane);
        {
            const int* src = reinterpret_cast<const int*>(desc + q);
            int* dst = reinterpret_cast<int*>(&sd);
            for (int i = lane; i < (int)(sizeof(BDesc) / 4); i += 32) dst[i] = __ldg(src + i);
        }
        __syncwarp();
        const int64_t first_item = __ldg(item_start + q);
        const int64_t b0 = (item - first_item) * bpi, b1 = min(sd.nb, b0 + bpi);
        Acc acc;
        acc.init();
        const int opc = sd.opc;
        if (opc == OPC_SUM) stream_bricks<Acc, OPC_SUM, BS>(c, sd, b0, b1, acc, lane);
        else if (opc == OPC_MIN) stream_bricks<Acc, OPC_MIN, BS>(c, sd, b0, b1, acc, lane);
        else stream_bricks<Acc, OPC_MAX, BS>(c, sd, b0, b1, acc, lane);
        long long s = acc.sum_bits();
        int32_t cmx = opc == OPC_MAX ? acc.code_max() : INT_MIN, cmn = opc == OPC_MIN ? ~acc.code_min() : INT_MIN;
#pragma unroll
        for (int o = 16; o; o >>= 1) s = SumOps<Acc>::add(s, __shfl_xor_sync(0xffffffffu, s, o));
        cmx = __reduce_max_sync(0xffffffffu, cmx);
        cmn = __reduce_max_sync(0xffffffffu, cmn);
        const int64_t nitems = (sd.nb + bpi - 1) / bpi;
        int last = 0;
        if (lane == 0) {
            item_sum[item] = s;
            item_ext[2 * item] = cmx;
            item_ext[2 * item + 1] = cmn;
            __threadfence();
            last = atomicAdd(done + q, 1) == (int)nitems - 1;
        }
        last = __shfl_sync(0xffffffffu, last, 0);
        if (last) {
            __threadfence();
            long long ts = 0;
            int32_t tmx = INT_MIN, tmn = INT_MIN;
            for (int64_t i = lane; i < nitems; i += 32) {
                const int64_t it = first_item + i;
                ts = SumOps<Acc>::add(ts, __ldcg(item_sum + it));
                tmx = max(tmx, __ldcg(item_ext + 2 * it));
                tmn = max(tmn, __ldcg(item_ext + 2 * it + 1));
            }
#pragma unroll
            for (int o = 16; o; o >>= 1) ts = SumOps<Acc>::add(ts, __shfl_xor_sync(0xffffffffu, ts, o));
            tmx = __reduce_max_sync(0xffffffffu, tmx);
            tmn = __reduce_max_sync(0xffffffffu, tmn);
            if (lane == 0) {
                psum[q] = ts;
                pext[2 * q] = tmx;
                pext[2 * q + 1] = tmn;
            }
        }
        __syncwarp();
    }
}

// ------------------------------------------------------------------ tile-shared scan

#include "tiles.cuh"

// ------------------------------------------------------------------ finalize / combine

__global__ void finalize_kernel(int nd, Extents ext, int dtype, int64_t nq, const olap_range* __restrict__ ranges,
                                const int32_t* __restrict__ ops, const int64_t* __restrict__ psum,
                                const int32_t* __restrict__ pext, olap_result* __restrict__ out) {
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nq; q += (int64_t)gridDim.x * blockDim.x) {
        olap_result r;
        r.i = 0;
        r.d = 0.0;
        r.flags = 0;
        r._pad = 0;
        const int32_t op = ops[q];
        bool invalid = op < OLAP_SUM || op > OLAP_AVG, empty = false;
        int64_t V = 1;
        for (int k = 0; k < nd; ++k) {
            const olap_range rg = ranges[q * nd + k];
            if (rg.lo < 0 || rg.hi >= ext.n[k]) invalid = true;
            if (rg.lo > rg.hi) empty = true;
            else V *= rg.hi - rg.lo + 1;
        }
        if (invalid) r.flags = OLAP_RESULT_INVALID;
        else if (empty) r.flags = OLAP_RESULT_EMPTY;
        else if (op == OLAP_COUNT) r.i = V;
        else {
            const int64_t s = psum[q];
            const int32_t cmx = pext[2 * q], cmn = ~pext[2 * q + 1];
            if (dtype == OLAP_INT32) {
                if (op == OLAP_SUM) r.i = s;
                else if (op == OLAP_MIN) r.i = cmn;
                else if (op == OLAP_MAX) r.i = cmx;
                else r.d = (double)s / (double)V;
            } else {
                const double ds = __longlong_as_double(s);
                if (op == OLAP_SUM) r.d = ds;
                else if (op == OLAP_MIN) r.d = (double)f32_decode(cmn);
                else if (op == OLAP_MAX) r.d = (double)f32_decode(cmx);
                else r.d = ds / (double)V;
            }
        }
        out[q] = r;
    }
}

__global__ void combine_kernel(int dtype, int64_t nq, const int64_t* __restrict__ s_in, const int32_t* __restrict__ e_in,
                               int64_t* s_acc, int32_t* e_acc) {
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nq; q += (int64_t)gridDim.x * blockDim.x) {
        if (dtype == OLAP_INT32)
            s_acc[q] = (int64_t)((uint64_t)s_acc[q] + (uint64_t)s_in[q]);
        else
            s_acc[q] = __double_as_longlong(__longlong_as_double(s_acc[q]) + __longlong_as_double(s_in[q]));
        e_acc[2 * q] = max(e_acc[2 * q], e_in[2 * q]);
        e_acc[2 * q + 1] = max(e_acc[2 * q + 1], e_in[2 * q + 1]);
    }
}

// ------------------------------------------------------------------ fill (support, not timed)

__device__ __forceinline__ uint64_t splitmix64_at(uint64_t seed, uint64_t idx) {
    uint64_t z = seed + (idx + 1ull) * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

struct FillParams {
    double c[kMaxDims + 1];
};

// Cell value of the global dim-0 row gr at logical offset off inside that row (the
// generators of olap_cube_fill, a function of the logical index only: layout-blind).
template <typename T>
__device__ __forceinline__ void gen_cell(T* cells, int64_t li, const Geo& geo, int gen, uint64_t seed,
                                         const FillParams& fp, int64_t gr, int64_t off) {
    if (gen == OLAP_GEN_UNIFORM) {
        const uint64_t z = splitmix64_at(seed, (uint64_t)(gr * geo.lrow + off));
        if (sizeof(T) == 4 && geo.dtype == OLAP_INT32)
            reinterpret_cast<int32_t*>(cells)[li] = (int32_t)(z >> 43) - (1 << 20);
        else
            reinterpret_cast<float*>(cells)[li] = (float)(z >> 40) * (1.0f / 16777216.0f);
    } else {
        double v = fp.c[0] + fp.c[1] * (double)gr;
        int64_t rem = off;
        for (int k = geo.nd - 1; k >= 1; --k) {
            const int64_t x = rem % geo.n[k];
            rem /= geo.n[k];
            v += fp.c[1 + k] * (double)x;
        }
        if (geo.dtype == OLAP_INT32) reinterpret_cast<int32_t*>(cells)[li] = (int32_t)v;
        else reinterpret_cast<float*>(cells)[li] = (float)v;
    }
}

template <typename T>
__global__ void fill_kernel(T* cells, Geo geo, int64_t row_cells, int gen, uint64_t seed, FillParams fp) {
    const int64_t n = geo.local_rows * row_cells;
    const int64_t ninner = geo.n[geo.nd - 1];
    for (int64_t li = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; li < n; li += (int64_t)gridDim.x * blockDim.x) {
        const int64_t lr = li / row_cells, poff = li - lr * row_cells;
        const int64_t rest = geo.nd > 1 ? poff / geo.pitch : 0, xin = poff - rest * geo.pitch;
        if (xin >= ninner) {  // padding cell: never part of a box
            cells[li] = (T)0;
            continue;
        }
        const int64_t off = rest * ninner + xin;  // logical offset inside the dim-0 row
        gen_cell<T>(cells, li, geo, gen, seed, fp, shard_global_of(lr, geo.G, geo.g, geo.b), off);
    }
}

// ------------------------------------------------------------------ bricked layouts (OLAP_LAYOUT_BRICK, _BRICK3)
// Cells (x_{N-3}, x_{N-2}, x_{N-1}) live in bricks of A0 x A x B = 32 cells (128 B: one DRAM fetch
// line on B200, profiles/r01/microbench_r01_sector.txt): 1 x 4 x 8 (OLAP_LAYOUT_BRICK) or 2 x 4 x 4
// (OLAP_LAYOUT_BRICK3).  The storage is the row-major array (x_0 .. x_{N-4}, W, X, Z, w, y, z) with
// x_{N-3} = A0 W + w, x_{N-2} = A X + y, x_{N-1} = B Z + z, held by an inner row-major cube of
// extents (.., NW, NX, NZ, 32); queries run brick_reduce_kernel on it (a lane quad per brick).
// When N = 3, x_{N-3} is dim 0 in SHARD-LOCAL rows (a query's owned rows are one local range), so
// a 2 x 4 x 4 brick pairs local rows 2W, 2W + 1 and the inner cube is the shard's own, unsharded.
struct BrickDims {
    int a0, a, b;
};
inline BrickDims brick_dims(int layout) { return layout == OLAP_LAYOUT_BRICK3 ? BrickDims{2, 4, 4} : BrickDims{1, 4, 8}; }

// olap_cube_fill on the brick array: storage index -> (leading, W, X, Z, w, y, z) -> logical cell.
template <typename T>
__global__ void fill_brick_kernel(T* cells, Geo geo, int64_t ncells, int64_t NW, int64_t NX, int64_t NZ, int a0, int a,
                                  int b, int64_t P1, int gen, uint64_t seed, FillParams fp) {
    const int nd = geo.nd;
    const int64_t na = geo.n[nd - 2], nb = geo.n[nd - 1], nw = nd == 3 ? geo.local_rows : geo.n[nd - 3];
    for (int64_t li = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; li < ncells; li += (int64_t)gridDim.x * blockDim.x) {
        const int c32 = (int)(li & 31);
        int64_t t = li >> 5;
        const int64_t Z = t % NZ;
        t /= NZ;
        const int64_t X = t % NX;
        t /= NX;
        const int64_t W = t % NW, mid = t / NW;
        const int64_t xw = a0 * W + c32 / (a * b), xa = a * X + (c32 / b) % a, xb = b * Z + c32 % b;
        if (xw >= nw || xa >= na || xb >= nb) {  // padding cell: never part of a box
            cells[li] = (T)0;
            continue;
        }
        int64_t lr, off;
        if (nd == 3) {
            lr = xw;
            off = xa * nb + xb;
        } else {  // mid = local row x P1 + the digits of dims 1..N-4
            lr = mid / P1;
            off = (((mid - lr * P1) * nw + xw) * na + xa) * nb + xb;
        }
        gen_cell<T>(cells, li, geo, gen, seed, fp, shard_global_of(lr, geo.G, geo.g, geo.b), off);
    }
}

// ------------------------------------------------------------------ build from facts (NEXT #2)

template <typename T>
__global__ void add_facts_kernel(T* cells, Geo geo, int64_t nrows, const int32_t* __restrict__ ids,
                                 const T* __restrict__ vals) {
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < nrows; r += (int64_t)gridDim.x * blockDim.x) {
        const int64_t x0 = ids[r];
        if (x0 < 0 || x0 >= geo.n[0]) continue;
        if (geo.G > 1 && (x0 / geo.b) % geo.G != geo.g) continue;  // row owned by another shard
        int64_t idx = shard_local_of(x0, geo.G, geo.b) * geo.stride[0];
        bool ok = true;
        for (int d = 1; d < geo.nd; ++d) {
            const int64_t x = ids[(int64_t)d * nrows + r];
            ok = ok && x >= 0 && x < geo.n[d];
            idx += x * geo.stride[d];
        }
        if (!ok) continue;
        atomicAdd(cells + idx, vals ? vals[r] : (T)1);
    }
}

// Deterministic float32 build: the cell each row adds into (local storage index), or kNoCell
// for rows another shard owns or with an id outside the cube; `row` = the row index (the sort's
// payload, so equal cells keep row order: the radix sort is stable).
constexpr unsigned long long kNoCell = ~0ull;
__global__ void fact_cell_kernel(Geo geo, int64_t nrows, const int32_t* __restrict__ ids, unsigned long long* key,
                                 int32_t* row) {
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < nrows; r += (int64_t)gridDim.x * blockDim.x) {
        const int64_t x0 = ids[r];
        bool ok = x0 >= 0 && x0 < geo.n[0] && (geo.G == 1 || (x0 / geo.b) % geo.G == geo.g);
        int64_t idx = ok ? shard_local_of(x0, geo.G, geo.b) * geo.stride[0] : 0;
        for (int d = 1; d < geo.nd; ++d) {
            const int64_t x = ids[(int64_t)d * nrows + r];
            ok = ok && x >= 0 && x < geo.n[d];
            idx += x * geo.stride[d];
        }
        key[r] = ok ? (unsigned long long)idx : kNoCell;
        row[r] = (int32_t)r;
    }
}

// One thread per run of equal cells in the sorted order (its head): the run's values are added in
// row order in fp64 and the cell gets (float)((double)cell + sum) -- one rounding per cell, the
// same sequence as oracle_factbuild, so the build is bit-exact and deterministic (no atomics).
__global__ void fact_segsum_kernel(float* cells, int64_t nrows, const unsigned long long* __restrict__ key,
                                   const int32_t* __restrict__ row, const float* __restrict__ vals) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nrows; i += (int64_t)gridDim.x * blockDim.x) {
        const unsigned long long k = key[i];
        if (k == kNoCell || (i > 0 && key[i - 1] == k)) continue;
        double acc = 0.0;
        for (int64_t j = i; j < nrows && key[j] == k; ++j) acc += vals ? (double)vals[row[j]] : 1.0;
        cells[k] = (float)((double)cells[k] + acc);
    }
}

}  // namespace olap

// ====================================================================== host runtime

using namespace olap;

struct olap_cube {
    int nd = 0, dtype = 0, device = 0;
    int64_t n[kMaxDims] = {};
    olap_shard sh{1, 0, 1};
    int64_t local_rows = 0, row_cells = 0, local_cells = 0;  // row_cells / local_cells include padding
    int64_t pitch = 0, lrow_cells = 0;                       // innermost pitch; logical cells per dim-0 row
    int64_t stride[kMaxDims] = {};
    void* d_cells = nullptr;

    std::mutex mu;
    cudaStream_t stream = nullptr;   // host-buffer calls
    cudaEvent_t ws_done = nullptr;   // last batch that used the workspace
    int num_sms = 0, blocks_per_sm = 0;

    int64_t nq_cap = 0, items_cap = 0;
    QDesc* d_desc = nullptr;
    int64_t* d_item_start = nullptr;
    int32_t* d_done = nullptr;
    int64_t* d_qtasks = nullptr;              // per query: tasks (planning scratch)
    int64_t* d_icnt = nullptr;                // per query: items (planning scratch, nq + 1)
    void* d_plantmp = nullptr;                // CUB scan scratch of the planners (item and pair offsets)
    size_t plan_bytes = 0;
    int32_t* d_qtv = nullptr;                 // per query: cells per task (planning scratch)
    unsigned long long* d_counter = nullptr;  // [0] item counter, [1] algorithmic bytes, [2..3] batch totals
    long long* d_item_sum = nullptr;
    int32_t* d_item_ext = nullptr;
    int32_t* d_order = nullptr;        // item execution order (L2-aware), items_cap entries
    int32_t* d_bucket = nullptr;       // bucket of every item, items_cap entries
    unsigned int* d_bcount = nullptr;  // [kMaxBuckets] counts + [kMaxBuckets] cursors
    int order_shift = -1;              // log2(bucket cells); -1: order disabled (cube fits in L2)
    // host-path staging
    olap_range* d_ranges = nullptr;
    int32_t* d_ops = nullptr;
    olap_result* d_results = nullptr;
    int64_t* d_psum = nullptr;
    int32_t* d_pext = nullptr;
    void* h_pinned = nullptr;
    size_t h_pinned_cap = 0;
    int64_t stage_cap = 0;

    // tile-shared scan (tiles.cuh): geometry, workspace, control words
    TGeo tg{};
    bool tiles_on = false;
    int64_t pairs_cap = 0, tq_cap = 0;
    TDesc* d_tdesc = nullptr;
    SDesc* d_sdesc = nullptr;
    int64_t* d_qpairs = nullptr;
    int64_t* d_pstart = nullptr;
    unsigned int* d_tcount = nullptr;  // ntiles + 1
    unsigned int* d_tstart = nullptr;  // ntiles + 1
    uint32_t* d_nonempty = nullptr;    // ntiles
    QDesc* d_tpds = nullptr;           // num_sms x kTileConsumers fallback descriptors of tile_reduce_kernel
    uint32_t* d_list = nullptr;        // pairs_cap
    long long* d_partial = nullptr;    // pairs_cap
    void* d_cubtmp = nullptr;
    size_t cub_bytes = 0;
    int32_t* d_ctl = nullptr;                  // [0] mode (1 = tiles), [1] non-empty tiles, [2] pop counter
    bool ctl_dirty = false;                    // a tile planner ran: d_ctl[0] may hold 1 (cleared when tiles go off)
    unsigned long long* d_ttot = nullptr;      // tile path batch totals (cells)

    bool prof = false;
    std::vector<cudaEvent_t> ev;
    size_t ev_used = 0;
    int64_t launches = 0;
    int64_t kernel_launches = 0;  // every kernel this cube launched (all entry points)
    unsigned long long bytes_base = 0;

    // OLAP_LAYOUT_BRICK / _BRICK3: this handle keeps the logical geometry (nd, n, shards) and
    // `inner` is the row-major cube of the brick array (.., NW, NX, NZ, 32) that owns the cells
    // (queries use its workspace: run_partials_brick).
    olap_cube* inner = nullptr;
    int brick_bps = 0;  // resident brick_reduce_kernel blocks per SM
    int layout = OLAP_LAYOUT_ROWMAJOR;  // OLAP_LAYOUT_BRICK / _BRICK3: `inner` holds the bricks

    // multi-GPU (mgpu.cu): a group handle (olap_cube_create_multi) owns `shards` (G shard cubes
    // over its devices) and answers through `exec`; a shard with an attached communicator
    // (olap_cube_attach_comm) answers through `exec` too; a plain cube builds `exec` lazily for
    // olap_query_stream.
    std::vector<olap_cube*> shards;
    olap::Exec* exec = nullptr;
    olap_comm* comm = nullptr;
    bool multi() const { return !shards.empty(); }

    // olap_query_batch on small batches replays a CUDA graph of its whole device sequence
    // (copy-in, plan, reduce, finalize, copy-out), one per batch size, captured on first use;
    // any workspace reallocation (ws_gen) invalidates them
    struct BatchGraph {
        int64_t nq = 0;
        uint64_t gen = 0, last = 0;
        int64_t kernels = 0, finals = 0;
        cudaGraphExec_t exec = nullptr;
    };
    std::vector<BatchGraph> graphs;
    uint64_t ws_gen = 0, graph_clock = 0;
};

namespace {

std::atomic<int64_t> g_finalize_launches{0};  // finalize is not bound to a cube (multi-GPU path)

struct DeviceGuard {
    int prev = -1;
    bool ok = false;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) == cudaSuccess && cudaSetDevice(dev) == cudaSuccess) ok = true;
    }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

Geo make_geo(const olap_cube* c) {
    Geo g;
    std::memset(&g, 0, sizeof(g));
    g.nd = c->nd;
    g.dtype = c->dtype;
    g.G = c->sh.nshards;
    g.g = c->sh.shard;
    g.b = c->sh.block;
    for (int k = 0; k < c->nd; ++k) {
        g.n[k] = c->n[k];
        g.stride[k] = c->stride[k];
    }
    g.local_rows = c->local_rows;
    g.pitch = c->pitch;
    g.lrow = c->lrow_cells;
    g.padded = c->pitch != c->n[c->nd - 1];
    return g;
}

void free_ws(olap_cube* c) {
    cudaFree(c->d_desc);
    cudaFree(c->d_item_start);
    cudaFree(c->d_done);
    cudaFree(c->d_qtasks);
    cudaFree(c->d_qtv);
    cudaFree(c->d_icnt);
    cudaFree(c->d_plantmp);
    c->d_qtasks = nullptr;
    c->d_qtv = nullptr;
    c->d_icnt = nullptr;
    c->d_plantmp = nullptr;
    c->plan_bytes = 0;
    cudaFree(c->d_item_sum);
    cudaFree(c->d_item_ext);
    cudaFree(c->d_order);
    cudaFree(c->d_bucket);
    cudaFree(c->d_bcount);
    c->d_order = nullptr;
    c->d_bucket = nullptr;
    c->d_bcount = nullptr;
    c->d_desc = nullptr;
    c->d_item_start = nullptr;
    c->d_done = nullptr;
    c->d_item_sum = nullptr;
    c->d_item_ext = nullptr;
    c->nq_cap = c->items_cap = 0;
    cudaFree(c->d_tdesc);
    cudaFree(c->d_sdesc);
    c->d_sdesc = nullptr;
    cudaFree(c->d_qpairs);
    cudaFree(c->d_pstart);
    cudaFree(c->d_tcount);
    cudaFree(c->d_tstart);
    cudaFree(c->d_nonempty);
    cudaFree(c->d_tpds);
    c->d_tpds = nullptr;
    cudaFree(c->d_list);
    cudaFree(c->d_partial);
    cudaFree(c->d_cubtmp);
    c->d_tdesc = nullptr;
    c->d_qpairs = c->d_pstart = nullptr;
    c->d_tcount = c->d_tstart = nullptr;
    c->d_nonempty = c->d_list = nullptr;
    c->d_partial = nullptr;
    c->d_cubtmp = nullptr;
    c->tq_cap = 0;
}

// Tile-path workspace (per query, per tile, per pair).  If it cannot be allocated the cube keeps
// answering through the item path (the tile path is an optimisation, never a requirement).
void ensure_tile_ws(olap_cube* c, int64_t cap) {
    if (!c->tiles_on || cap <= c->tq_cap) return;
    const int64_t nt = c->tg.ntiles;
    // test hook: simulate an allocation failure above a query capacity (tests/test_gpu_tiles.py)
    const char* lim = getenv("OLAP_TEST_TILE_WS_LIMIT");
    bool ok = !(lim && cap > atoll(lim)) && cudaMalloc(&c->d_tdesc, sizeof(TDesc) * cap) == cudaSuccess &&
              cudaMalloc(&c->d_sdesc, sizeof(SDesc) * cap) == cudaSuccess &&
              cudaMalloc(&c->d_qpairs, sizeof(int64_t) * (cap + 1)) == cudaSuccess &&
              cudaMalloc(&c->d_pstart, sizeof(int64_t) * (cap + 1)) == cudaSuccess;
    if (ok && !c->d_tcount) {
        ok = cudaMalloc(&c->d_tcount, sizeof(unsigned int) * (3 * nt + 1)) == cudaSuccess &&
             cudaMalloc(&c->d_tstart, sizeof(unsigned int) * (3 * nt + 1)) == cudaSuccess &&
             cudaMalloc(&c->d_nonempty, sizeof(uint32_t) * nt) == cudaSuccess &&
             cudaMalloc(&c->d_tpds, sizeof(QDesc) * (size_t)c->num_sms * kTileConsumers) == cudaSuccess &&
             cudaMalloc(&c->d_list, sizeof(uint32_t) * c->pairs_cap) == cudaSuccess &&
             cudaMalloc(&c->d_partial, sizeof(long long) * c->pairs_cap) == cudaSuccess;
        if (ok) {
            c->cub_bytes = 0;
            ok = cub::DeviceScan::ExclusiveSum(nullptr, c->cub_bytes, c->d_tcount, c->d_tstart, (int)(3 * nt + 1)) ==
                     cudaSuccess &&
                 cudaMalloc(&c->d_cubtmp, std::max<size_t>(c->cub_bytes, 16)) == cudaSuccess;
        }
    }
    if (!ok) {
        cudaGetLastError();
        c->tiles_on = false;  // free_ws releases whatever was allocated
        return;
    }
    c->tq_cap = cap;
}

int ensure_ws(olap_cube* c, int64_t nq) {
    if (nq <= c->nq_cap) return OLAP_OK;
    OLAP_CUDA_TRY(cudaEventSynchronize(c->ws_done));
    ++c->ws_gen;
    free_ws(c);
    int64_t cap = std::max<int64_t>(nq, 1024);
    // item partial capacity: >= 2^20 and 4 per query, and for big cubes enough that items stay a
    // few MiB (the L2-aware order needs the ~600 in-flight items to fit in L2): one per 4 KiB of
    // cube, <= 2^24 (a batch reads the cube ~10^2-10^3 times over at C3-like overlap)
    const int64_t by_size = std::min<int64_t>(1ll << 24, (c->local_cells * 4) >> 12);
    int64_t items = std::max<int64_t>(std::max<int64_t>(1ll << 20, 4 * cap), by_size);
    OLAP_CUDA_TRY(cudaMalloc(&c->d_desc, sizeof(QDesc) * cap));
    OLAP_CUDA_TRY(cudaMalloc(&c->d_item_start, sizeof(int64_t) * (cap + 1)));
    OLAP_CUDA_TRY(cudaMalloc(&c->d_done, sizeof(int32_t) * cap));
    OLAP_CUDA_TRY(cudaMalloc(&c->d_qtasks, sizeof(int64_t) * cap));
    OLAP_CUDA_TRY(cudaMalloc(&c->d_qtv, sizeof(int32_t) * cap));
    OLAP_CUDA_TRY(cudaMalloc(&c->d_icnt, sizeof(int64_t) * (cap + 2)));
    c->plan_bytes = 0;
    OLAP_CUDA_TRY(cub::DeviceScan::ExclusiveSum(nullptr, c->plan_bytes, c->d_icnt, c->d_item_start, (int)(cap + 1)));
    OLAP_CUDA_TRY(cudaMalloc(&c->d_plantmp, std::max<size_t>(c->plan_bytes, 16)));
    OLAP_CUDA_TRY(cudaMalloc(&c->d_item_sum, sizeof(long long) * items));
    OLAP_CUDA_TRY(cudaMalloc(&c->d_item_ext, sizeof(int32_t) * 2 * items));
    if (c->order_shift >= 0) {
        OLAP_CUDA_TRY(cudaMalloc(&c->d_order, sizeof(int32_t) * items));
        OLAP_CUDA_TRY(cudaMalloc(&c->d_bucket, sizeof(int32_t) * items));
        OLAP_CUDA_TRY(cudaMalloc(&c->d_bcount, sizeof(unsigned int) * 2 * kMaxBuckets));
    }
    c->nq_cap = cap;
    c->items_cap = items;
    ensure_tile_ws(c, cap);
    return OLAP_OK;
}

int ensure_stage(olap_cube* c, int64_t nq) {
    if (nq <= c->stage_cap) return OLAP_OK;
    OLAP_CUDA_TRY(cudaEventSynchronize(c->ws_done));
    ++c->ws_gen;
    cudaFree(c->d_ranges);
    cudaFree(c->d_ops);
    cudaFree(c->d_results);
    cudaFree(c->d_psum);
    cudaFree(c->d_pext);
    cudaFreeHost(c->h_pinned);
    c->d_ranges = nullptr;
    c->d_ops = nullptr;
    c->d_results = nullptr;
    c->d_psum = nullptr;
    c->d_pext = nullptr;
    c->h_pinned = nullptr;
    c->stage_cap = 0;
    int64_t cap = std::max<int64_t>(nq, 1024);
    OLAP_CUDA_TRY(cudaMalloc(&c->d_ranges, sizeof(olap_range) * c->nd * cap));
    OLAP_CUDA_TRY(cudaMalloc(&c->d_ops, sizeof(int32_t) * cap));
    OLAP_CUDA_TRY(cudaMalloc(&c->d_results, sizeof(olap_result) * cap));
    OLAP_CUDA_TRY(cudaMalloc(&c->d_psum, sizeof(int64_t) * cap));
    OLAP_CUDA_TRY(cudaMalloc(&c->d_pext, sizeof(int32_t) * 2 * cap));
    c->h_pinned_cap = (sizeof(olap_range) * c->nd + sizeof(int32_t) + sizeof(olap_result)) * cap;
    OLAP_CUDA_TRY(cudaHostAlloc(&c->h_pinned, c->h_pinned_cap, cudaHostAllocDefault));
    c->stage_cap = cap;
    return OLAP_OK;
}

// plan + reduce for nq queries already on the device; writes partials
bool capturing(cudaStream_t st) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    return cudaStreamIsCapturing(st, &cs) == cudaSuccess && cs == cudaStreamCaptureStatusActive;
}

// plan + reduce for nq queries already on the device; writes partials.  Capturable into a
// CUDA graph once the workspace has grown to nq (a warm-up call outside capture): inside a
// capture the cross-stream workspace event and the profiling events are left out.
int run_partials_brick(olap_cube* c, int64_t nq, const olap_range* d_ranges, const int32_t* d_ops, int64_t* d_psum,
                       int32_t* d_pext, cudaStream_t st);

int run_partials(olap_cube* c, int64_t nq, const olap_range* d_ranges, const int32_t* d_ops, int64_t* d_psum,
                 int32_t* d_pext, cudaStream_t st) {
    if (c->inner) return run_partials_brick(c, nq, d_ranges, d_ops, d_psum, d_pext, st);
    const bool cap = capturing(st);
    if (cap && nq > c->nq_cap)
        return set_error(OLAP_E_STATE, "stream capture: run one batch of %lld queries outside capture first "
                         "(the workspace cannot grow inside a CUDA graph)", (long long)nq);
    int rc = ensure_ws(c, nq);
    if (rc) return rc;
    if (!cap) OLAP_CUDA_TRY(cudaStreamWaitEvent(st, c->ws_done, 0));
    const bool prof = c->prof && !cap;
    auto bracket = [&](cudaEvent_t* e0, cudaEvent_t* e1) -> int {
        while (c->ev.size() < c->ev_used + 2) {
            cudaEvent_t e;
            OLAP_CUDA_TRY(cudaEventCreate(&e));
            c->ev.push_back(e);
        }
        *e0 = c->ev[c->ev_used];
        *e1 = c->ev[c->ev_used + 1];
        c->ev_used += 2;
        return OLAP_OK;
    };
    const int32_t* tmode = c->d_ctl;  // stays 0 when the cube has no tile path
    if (!c->tiles_on && c->ctl_dirty) {
        // the tile path was switched off (workspace growth failed) after a batch that took it:
        // clear the stale mode word, or every item-path kernel below would return at once
        OLAP_CUDA_TRY(cudaMemsetAsync(c->d_ctl, 0, sizeof(int32_t), st));
        c->ctl_dirty = false;
    }
    if (c->tiles_on) {
        c->ctl_dirty = true;
        // tile-shared scan (tiles.cuh); tile_scan_kernel picks it or the item path on the device
        const TGeo& tg = c->tg;
        const int qb = (int)((nq + kDescThreads - 1) / kDescThreads), eg = c->num_sms * 8;
        OLAP_CUDA_TRY(cudaMemsetAsync(c->d_ttot, 0, sizeof(unsigned long long), st));
        tile_desc_kernel<<<qb, kDescThreads, 0, st>>>(make_geo(c), tg, nq, d_ranges, d_ops, c->d_tdesc, c->d_sdesc,
                                                      c->d_qpairs,
                                                      d_psum, d_pext, c->d_ttot);
        OLAP_CUDA_TRY(cudaMemsetAsync(c->d_qpairs + nq, 0, sizeof(int64_t), st));
        size_t pb = c->plan_bytes;
        OLAP_CUDA_TRY(cub::DeviceScan::ExclusiveSum(c->d_plantmp, pb, c->d_qpairs, c->d_pstart, (int)(nq + 1), st));
        tile_scan_kernel<<<1, 1, 0, st>>>(c->d_pstart, nq, c->pairs_cap, tg, c->d_ttot, c->d_ctl, c->d_counter + 1);
        OLAP_CUDA_TRY(cudaMemsetAsync(c->d_tcount, 0, sizeof(unsigned int) * (3 * tg.ntiles + 1), st));
        tile_count_kernel<<<eg, 256, 0, st>>>(tg, nq, c->d_pstart, c->d_tdesc, c->d_tcount, c->d_ctl);
        OLAP_CUDA_TRY(cudaGetLastError());
        size_t tb = c->cub_bytes;
        OLAP_CUDA_TRY(cub::DeviceScan::ExclusiveSum(c->d_cubtmp, tb, c->d_tcount, c->d_tstart,
                                                    (int)(3 * tg.ntiles + 1), st));
        tile_compact_kernel<<<eg, 256, 0, st>>>(tg.ntiles, c->d_tstart, c->d_ctl, c->d_nonempty);
        tile_scatter_kernel<<<eg, 256, 0, st>>>(tg, nq, c->d_pstart, c->d_tdesc, c->d_tcount, c->d_tstart, c->d_ctl,
                                                c->d_list);
        cudaEvent_t t0 = nullptr, t1 = nullptr;
        if (prof) {
            int rc2 = bracket(&t0, &t1);
            if (rc2) return rc2;
            OLAP_CUDA_TRY(cudaEventRecord(t0, st));
        }
        if (c->dtype == OLAP_INT32)
            tile_reduce_kernel<int32_t, AccI><<<c->num_sms, kTileThreads, tile_smem_bytes<AccI>(), st>>>(
                static_cast<const int32_t*>(c->d_cells), tg, c->d_tdesc, c->d_sdesc, c->d_pstart, c->d_tstart,
                c->d_nonempty, c->d_list, c->d_ctl, c->d_partial, c->d_tpds);
        else
            tile_reduce_kernel<float, AccF><<<c->num_sms, kTileThreads, tile_smem_bytes<AccF>(), st>>>(
                static_cast<const float*>(c->d_cells), tg, c->d_tdesc, c->d_sdesc, c->d_pstart, c->d_tstart,
                c->d_nonempty, c->d_list, c->d_ctl, c->d_partial, c->d_tpds);
        OLAP_CUDA_TRY(cudaGetLastError());
        if (prof) OLAP_CUDA_TRY(cudaEventRecord(t1, st));
        const int fg = (int)std::min<int64_t>(nq, (int64_t)c->num_sms * 8);
        if (c->dtype == OLAP_INT32)
            pair_fold_kernel<AccI><<<fg, 256, 0, st>>>(nq, c->d_pstart, c->d_tdesc, c->d_ctl, c->d_partial, d_psum,
                                                       d_pext);
        else
            pair_fold_kernel<AccF><<<fg, 256, 0, st>>>(nq, c->d_pstart, c->d_tdesc, c->d_ctl, c->d_partial, d_psum,
                                                       d_pext);
        OLAP_CUDA_TRY(cudaGetLastError());
        c->kernel_launches += 11;  // desc, CUB scan (2), choice, count, CUB scan (2), compact, scatter, reduce, fold
    }
    OLAP_CUDA_TRY(cudaMemsetAsync(c->d_counter + 2, 0, 2 * sizeof(unsigned long long), st));
    desc_kernel<<<(int)((nq + kDescThreads - 1) / kDescThreads), kDescThreads, 0, st>>>(
        make_geo(c), nq, d_ranges, d_ops, c->d_desc, c->d_qtasks, c->d_qtv, c->d_done, d_psum, d_pext, c->d_counter + 2,
        tmode);
    OLAP_CUDA_TRY(cudaGetLastError());
    const int grid = c->num_sms * c->blocks_per_sm;
    const bool witems = kWarpItemsMode >= 0 ? kWarpItemsMode != 0 : nq > kWarpItemQueries * grid;
    if (nq <= kPlanSmall) {
        plan_small_kernel<<<1, kPlanThreads, 0, st>>>(nq, c->d_desc, c->d_qtasks, c->d_qtv, c->d_item_start,
                                                      c->d_counter, c->items_cap, c->d_counter + 2, c->d_counter + 1,
                                                      grid, witems ? 1 : 0, tmode);
        OLAP_CUDA_TRY(cudaGetLastError());
        c->kernel_launches -= 3;
    } else {
        items_kernel<<<(int)((nq + kDescThreads) / kDescThreads), kDescThreads, 0, st>>>(
            nq, c->d_desc, c->d_qtasks, c->d_qtv, c->d_icnt, c->items_cap, c->d_counter + 2, grid, witems ? 1 : 0,
            tmode);
        OLAP_CUDA_TRY(cudaGetLastError());
        size_t pb = c->plan_bytes;
        OLAP_CUDA_TRY(cub::DeviceScan::ExclusiveSum(c->d_plantmp, pb, c->d_icnt, c->d_item_start, (int)(nq + 1), st));
        scan_fix_kernel<<<1, 1, 0, st>>>(nq, c->d_item_start, c->d_counter, c->items_cap, c->d_counter + 2,
                                         c->d_counter + 1, tmode);
        OLAP_CUDA_TRY(cudaGetLastError());
    }
    const int32_t* order = nullptr;
    c->kernel_launches += 6;  // desc, items, CUB scan (2), scan_fix, reduce
    if (c->order_shift >= 0) {
        c->kernel_launches += 3;
        OLAP_CUDA_TRY(cudaMemsetAsync(c->d_bcount, 0, sizeof(unsigned int) * kMaxBuckets, st));
        bucket_kernel<<<c->num_sms * 8, 256, 0, st>>>(nq, c->d_desc, c->d_item_start, c->order_shift, c->d_bucket,
                                                       c->d_bcount, tmode);
        bucket_scan_kernel<<<1, 1024, 0, st>>>(c->d_bcount, c->d_bcount + kMaxBuckets, tmode);
        scatter_kernel<<<c->num_sms * 8, 256, 0, st>>>(nq, c->d_item_start, c->d_bucket, c->d_bcount + kMaxBuckets,
                                                        c->d_order, tmode);
        OLAP_CUDA_TRY(cudaGetLastError());
        order = c->d_order;
    }
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    if (prof) {
        int rc2 = bracket(&e0, &e1);
        if (rc2) return rc2;
        OLAP_CUDA_TRY(cudaEventRecord(e0, st));
    }
    if (witems) {
        if (c->dtype == OLAP_INT32)
            reduce_kernel_w<int32_t, AccI><<<grid, kThreads, 0, st>>>(
                static_cast<const int32_t*>(c->d_cells), nq, c->d_desc, c->d_item_start, c->d_counter, c->d_done,
                c->d_item_sum, c->d_item_ext, d_psum, d_pext, order, tmode);
        else
            reduce_kernel_w<float, AccF><<<grid, kThreads, 0, st>>>(
                static_cast<const float*>(c->d_cells), nq, c->d_desc, c->d_item_start, c->d_counter, c->d_done,
                c->d_item_sum, c->d_item_ext, d_psum, d_pext, order, tmode);
    } else if (c->dtype == OLAP_INT32)
        reduce_kernel<int32_t, AccI><<<grid, kThreads, 0, st>>>(
            static_cast<const int32_t*>(c->d_cells), nq, c->d_desc, c->d_item_start, c->d_counter, c->d_done,
            c->d_item_sum, c->d_item_ext, d_psum, d_pext, order, tmode);
    else
        reduce_kernel<float, AccF><<<grid, kThreads, 0, st>>>(
            static_cast<const float*>(c->d_cells), nq, c->d_desc, c->d_item_start, c->d_counter, c->d_done,
            c->d_item_sum, c->d_item_ext, d_psum, d_pext, order, tmode);
    OLAP_CUDA_TRY(cudaGetLastError());
    if (prof) {
        OLAP_CUDA_TRY(cudaEventRecord(e1, st));
        ++c->launches;
    }
    if (!cap) OLAP_CUDA_TRY(cudaEventRecord(c->ws_done, st));
    return OLAP_OK;
}

int launch_finalize(int nd, const int64_t* ext, int dtype, int64_t nq, const olap_range* d_ranges, const int32_t* d_ops,
                    const int64_t* d_psum, const int32_t* d_pext, olap_result* d_results, cudaStream_t st) {
    Extents e;
    std::memset(&e, 0, sizeof(e));
    for (int k = 0; k < nd; ++k) e.n[k] = ext[k];
    const int grid = (int)std::min<int64_t>((nq + 255) / 256, 4096);
    g_finalize_launches.fetch_add(1);
    finalize_kernel<<<grid, 256, 0, st>>>(nd, e, dtype, nq, d_ranges, d_ops, d_psum, d_pext, d_results);
    OLAP_CUDA_TRY(cudaGetLastError());
    return OLAP_OK;
}

// Bricked cube: plan (brick_desc_kernel, brick_items_kernel, CUB scan) and reduce
// (brick_reduce_kernel) on the inner cube's workspace.
int run_partials_brick(olap_cube* c, int64_t nq, const olap_range* d_ranges, const int32_t* d_ops, int64_t* d_psum,
                       int32_t* d_pext, cudaStream_t st) {
    olap_cube* ic = c->inner;
    const bool cap = capturing(st);
    if (cap && nq > ic->nq_cap)
        return set_error(OLAP_E_STATE, "stream capture: run one batch of %lld queries outside capture first "
                         "(the workspace cannot grow inside a CUDA graph)", (long long)nq);
    int rc = ensure_ws(ic, nq);
    if (rc) return rc;
    if (!cap) OLAP_CUDA_TRY(cudaStreamWaitEvent(st, ic->ws_done, 0));
    BGeo g;
    std::memset(&g, 0, sizeof(g));
    g.nd = c->nd;
    g.G = c->sh.nshards;
    g.g = c->sh.shard;
    g.b = c->sh.block;
    for (int k = 0; k < c->nd; ++k) g.n[k] = c->n[k];
    for (int k = 0; k <= c->nd - 2; ++k) g.stride[k] = ic->stride[k];
    g.local_rows = c->local_rows;
    BDesc* bd = reinterpret_cast<BDesc*>(ic->d_desc);
    const bool b3 = c->layout == OLAP_LAYOUT_BRICK3;
    if (!c->brick_bps) {
        int bps = 0;
        if (c->dtype == OLAP_INT32)
            OLAP_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(
                &bps, b3 ? brick_reduce_kernel<int32_t, AccI, 1> : brick_reduce_kernel<int32_t, AccI, 0>, kThreads, 0));
        else
            OLAP_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(
                &bps, b3 ? brick_reduce_kernel<float, AccF, 1> : brick_reduce_kernel<float, AccF, 0>, kThreads, 0));
        c->brick_bps = std::max(bps, 1);
    }
    const int grid = ic->num_sms * c->brick_bps;
    OLAP_CUDA_TRY(cudaMemsetAsync(ic->d_counter + 2, 0, 2 * sizeof(unsigned long long), st));
    (b3 ? brick_desc_kernel<1> : brick_desc_kernel<0>)<<<(int)((nq + 255) / 256), 256, 0, st>>>(
        g, nq, d_ranges, d_ops, bd, ic->d_qtasks, ic->d_done, d_psum, d_pext, ic->d_counter + 2);
    brick_items_kernel<<<(int)((nq + 256) / 256), 256, 0, st>>>(nq, bd, ic->d_qtasks, ic->d_icnt, ic->items_cap,
                                                                ic->d_counter + 2, grid * kWarps);
    OLAP_CUDA_TRY(cudaGetLastError());
    size_t pb = ic->plan_bytes;
    OLAP_CUDA_TRY(cub::DeviceScan::ExclusiveSum(ic->d_plantmp, pb, ic->d_icnt, ic->d_item_start, (int)(nq + 1), st));
    scan_fix_kernel<<<1, 1, 0, st>>>(nq, ic->d_item_start, ic->d_counter, ic->items_cap, ic->d_counter + 2,
                                     ic->d_counter + 1, nullptr);
    OLAP_CUDA_TRY(cudaGetLastError());
    const bool prof = ic->prof && !cap;
    if (prof) {
        while (ic->ev.size() < ic->ev_used + 2) {
            cudaEvent_t e;
            OLAP_CUDA_TRY(cudaEventCreate(&e));
            ic->ev.push_back(e);
        }
        OLAP_CUDA_TRY(cudaEventRecord(ic->ev[ic->ev_used], st));
    }
    if (c->dtype == OLAP_INT32)
        (b3 ? brick_reduce_kernel<int32_t, AccI, 1> : brick_reduce_kernel<int32_t, AccI, 0>)<<<grid, kThreads, 0, st>>>(
            static_cast<const int32_t*>(ic->d_cells), nq, bd, ic->d_item_start, ic->d_icnt, ic->d_counter, ic->d_done,
            ic->d_item_sum, ic->d_item_ext, d_psum, d_pext);
    else
        (b3 ? brick_reduce_kernel<float, AccF, 1> : brick_reduce_kernel<float, AccF, 0>)<<<grid, kThreads, 0, st>>>(
            static_cast<const float*>(ic->d_cells), nq, bd, ic->d_item_start, ic->d_icnt, ic->d_counter, ic->d_done,
            ic->d_item_sum, ic->d_item_ext, d_psum, d_pext);
    OLAP_CUDA_TRY(cudaGetLastError());
    if (prof) {
        OLAP_CUDA_TRY(cudaEventRecord(ic->ev[ic->ev_used + 1], st));
        ic->ev_used += 2;
        ++ic->launches;
    }
    c->kernel_launches += 6;  // desc, items, CUB scan (2), fix, reduce
    if (!cap) {
        OLAP_CUDA_TRY(cudaEventRecord(ic->ws_done, st));
        OLAP_CUDA_TRY(cudaEventRecord(c->ws_done, st));
    }
    return OLAP_OK;
}

// Host rows [row_lo, row_hi) (logical row-major) -> brick order, one dim-0 row at a time.  A row is
// one inner row, except for 2 x 4 x 4 bricks of a 3-D cube: there local rows 2W and 2W + 1 share
// inner row W, each holding the first or second 16-cell half of every brick (one strided copy).
int load_rows_brick(olap_cube* c, int64_t row_lo, int64_t row_hi, const void* cells) {
    olap_cube* ic = c->inner;
    const int nd = c->nd;
    const BrickDims bd = brick_dims(c->layout);
    const int64_t na = c->n[nd - 2], nb = c->n[nd - 1];
    const int64_t NW = ic->n[nd - 3], NX = ic->n[nd - 2], NZ = ic->n[nd - 1];
    const bool pair_rows = nd == 3 && bd.a0 == 2;
    const int64_t nw = nd == 3 ? 1 : c->n[nd - 3];         // x_{N-3} values inside one dim-0 row
    const int64_t P1 = nd == 3 ? 1 : c->lrow_cells / (nw * na * nb);  // digits of dims 1..N-4
    const int64_t half = 32 / bd.a0;                        // cells of one x_{N-3} layer of a brick
    const int64_t bufcells = pair_rows ? NX * NZ * half : ic->row_cells;
    std::vector<uint32_t> buf;
    try {
        buf.assign((size_t)bufcells, 0u);
    } catch (...) {
        return set_error(OLAP_E_NOMEM, "host staging of one brick row (%lld cells)", (long long)bufcells);
    }
    const uint32_t* src = static_cast<const uint32_t*>(cells);
    char* dst = static_cast<char*>(ic->d_cells);
    const int64_t G = c->sh.nshards, g = c->sh.shard, b = c->sh.block;
    for (int64_t r = row_lo; r < row_hi; ++r) {
        if (G > 1 && (r / b) % G != g) continue;
        const uint32_t* row = src + (r - row_lo) * c->lrow_cells;
        for (int64_t mid = 0; mid < P1; ++mid)
            for (int64_t xw = 0; xw < nw; ++xw)
                for (int64_t xa = 0; xa < na; ++xa) {
                    const uint32_t* in = row + ((mid * nw + xw) * na + xa) * nb;
                    // brick (W, X, Z) of this row and the cell's place inside it
                    const int64_t W = nd == 3 ? 0 : mid * NW + xw / bd.a0;
                    const int64_t wofs = nd == 3 ? 0 : (xw % bd.a0) * half;
                    uint32_t* out = buf.data() + ((W * NX + xa / bd.a) * NZ) * (pair_rows ? half : 32) + wofs +
                                    (xa % bd.a) * bd.b;
                    for (int64_t xb = 0; xb < nb; ++xb) out[(xb / bd.b) * (pair_rows ? half : 32) + xb % bd.b] = in[xb];
                }
        const int64_t lr = shard_local_of(r, G, b);
        if (pair_rows)  // half-bricks: 64 B of every 128-B brick of inner row lr / 2
            OLAP_CUDA_TRY(cudaMemcpy2D(dst + ((lr >> 1) * ic->row_cells + (lr & 1) * half) * 4, 128, buf.data(),
                                       half * 4, half * 4, NX * NZ, cudaMemcpyHostToDevice));
        else
            OLAP_CUDA_TRY(cudaMemcpy(dst + lr * ic->row_cells * 4, buf.data(), ic->row_cells * 4, cudaMemcpyHostToDevice));
    }
    return OLAP_OK;
}

// Tile geometry (tiles.cuh): kt = outermost dim whose stride fits a 64 KiB tile; a tile is ct
// consecutive indices of dim kt times everything inside it (contiguous, and a box).  The tile
// path is enabled for cubes that do not fit in L2 (the item path already serves those from L2).
void make_tiles(olap_cube* c) {
    TGeo& t = c->tg;
    std::memset(&t, 0, sizeof(t));
    const int nd = c->nd;
    t.nd = nd;
    t.padded = c->pitch != c->n[nd - 1];
    for (int k = 0; k < nd; ++k) {
        t.ext[k] = k == 0 ? c->local_rows : c->n[k];
        t.stride[k] = nd == 1 ? 1 : c->stride[k];
    }
    int kt = 0;
    const int64_t tcap = tile_cells_max(c->dtype == OLAP_FLOAT32);
    while (t.stride[kt] > tcap) ++kt;
    t.kt = kt;
    int64_t ctmax = std::max<int64_t>(1, tcap / t.stride[kt]);
    const int64_t ekt = std::max<int64_t>(t.ext[kt], 1);
    const int64_t nch = (ekt + ctmax - 1) / ctmax;
    int64_t ct = (ekt + nch - 1) / nch;
    if (kt == nd - 1) ct = (ct + 7) & ~7ll;  // chunks of the innermost row start 32-B aligned
    t.ct = ct;
    t.nct = (ekt + ct - 1) / ct;
    t.ts[kt] = 1;
    for (int e = kt - 1; e >= 0; --e) t.ts[e] = t.ts[e + 1] * (e + 1 == kt ? t.nct : t.ext[e + 1]);
    t.ntiles = t.ts[0] * (kt == 0 ? t.nct : t.ext[0]);
    t.tcells = ct * t.stride[kt];
    t.ok = c->local_rows > 0 && t.ntiles < (1ll << 31) && c->order_shift >= 0 && !getenv("OLAP_NO_TILES");
    c->tiles_on = t.ok;
    c->pairs_cap = std::min<int64_t>(1ll << 29, std::max<int64_t>(1ll << 24, c->local_cells / 8));
    if (c->tiles_on) {
        if (cudaFuncSetAttribute(tile_reduce_kernel<int32_t, AccI>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)tile_smem_bytes<AccI>()) != cudaSuccess ||
            cudaFuncSetAttribute(tile_reduce_kernel<float, AccF>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)tile_smem_bytes<AccF>()) != cudaSuccess) {
            cudaGetLastError();
            c->tiles_on = false;
            t.ok = 0;
        }
    }
}

int check_cube(const olap_cube* c) {
    if (!c) return set_error(OLAP_E_INVALID, "cube handle is NULL");
    if (c->multi()) return OLAP_OK;
    if (!c->d_cells) return set_error(OLAP_E_STATE, "cube has no device storage");
    return OLAP_OK;
}

}  // namespace

namespace olap {
// geometry for other translation units (hier.cu): dims, extents, dtype, inner pitch, shards
int cube_geometry(const olap_cube* c, int* nd, int64_t* n, int* dtype, int64_t* pitch, int64_t* nshards) {
    *nd = c->nd;
    for (int k = 0; k < c->nd; ++k) n[k] = c->n[k];
    *dtype = c->dtype;
    *pitch = c->pitch;
    *nshards = c->sh.nshards;
    return OLAP_OK;
}
// OLAP_LAYOUT_ROWMAJOR, _BRICK or _BRICK3 (roll-up reads raw cells and needs row-major)
int cube_layout(const olap_cube* c) { return c->layout; }
}  // namespace olap

extern "C" {

int olap_cube_create(int ndims, const int64_t* extents, int dtype, const olap_shard* shard, int device,
                     olap_cube** out) {
    clear_error();
    if (!out || !extents) return set_error(OLAP_E_INVALID, "olap_cube_create: NULL argument");
    if (ndims < 1 || ndims > kMaxDims) return set_error(OLAP_E_INVALID, "ndims %d not in [1,8]", ndims);
    if (dtype != OLAP_INT32 && dtype != OLAP_FLOAT32) return set_error(OLAP_E_INVALID, "bad dtype %d", dtype);
    olap_shard sh{1, 0, 1};
    if (shard) sh = *shard;
    if (sh.nshards < 1 || sh.shard < 0 || sh.shard >= sh.nshards || sh.block < 1)
        return set_error(OLAP_E_INVALID, "bad shard {%lld,%lld,%lld}", (long long)sh.nshards, (long long)sh.shard,
                         (long long)sh.block);
    int64_t cells = 1;
    for (int k = 0; k < ndims; ++k) {
        if (extents[k] < 1) return set_error(OLAP_E_INVALID, "extent[%d] = %lld < 1", k, (long long)extents[k]);
        if (extents[k] > kMaxExtent)
            return set_error(OLAP_E_UNSUPPORTED, "extent[%d] = %lld exceeds 2^30", k, (long long)extents[k]);
        cells *= extents[k];
        if (cells > kMaxCells) return set_error(OLAP_E_UNSUPPORTED, "cube exceeds 2^42 cells");
    }
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
        return set_error(OLAP_E_CUDA, "no CUDA device available (the library has no CPU fallback)");
    if (device < 0 || device >= ndev) return set_error(OLAP_E_INVALID, "device %d not in [0,%d)", device, ndev);
    DeviceGuard dg(device);
    if (!dg.ok) return set_error(OLAP_E_CUDA, "cudaSetDevice(%d) failed", device);

    olap_cube* c = new (std::nothrow) olap_cube();
    if (!c) return set_error(OLAP_E_NOMEM, "host allocation failed");
    c->nd = ndims;
    c->dtype = dtype;
    c->device = device;
    c->sh = sh;
    for (int k = 0; k < ndims; ++k) c->n[k] = extents[k];
    // innermost pitch padded to a multiple of 4 cells (16 B) when needed so that every
    // innermost row starts 16-B aligned for the vector path
    // (8 cells = 32 B for LDG.256 slots when the extent is >= 32, so padding stays <= 22%)
    c->pitch = c->n[ndims - 1];
    if (ndims > 1 && c->pitch >= 32 && (c->pitch & 7)) c->pitch = (c->pitch + 7) & ~7ll;
    else if (ndims > 1 && (c->pitch & 3)) c->pitch = (c->pitch + 3) & ~3ll;
    c->stride[ndims - 1] = 1;
    for (int k = ndims - 2; k >= 0; --k) c->stride[k] = c->stride[k + 1] * (k == ndims - 2 ? c->pitch : c->n[k + 1]);
    c->row_cells = ndims > 1 ? c->stride[0] : 1;
    c->lrow_cells = 1;
    for (int k = 1; k < ndims; ++k) c->lrow_cells *= c->n[k];
    c->local_rows = shard_rows(c->n[0], sh.nshards, sh.shard, sh.block);
    c->local_cells = c->local_rows * c->row_cells;
    int rc = OLAP_OK;
    // +64 B: a run's last 32-B slot may extend up to 7 cells past the final cell (masked)
    cudaError_t e = cudaMalloc(&c->d_cells, std::max<int64_t>(c->local_cells, 1) * 4 + 64);
    if (e != cudaSuccess) {
        rc = set_error(e == cudaErrorMemoryAllocation ? OLAP_E_NOMEM : OLAP_E_CUDA, "cudaMalloc of %lld cells: %s",
                       (long long)c->local_cells, cudaGetErrorString(e));
        cudaGetLastError();
        delete c;
        return rc;
    }
    if (c->pitch != c->n[ndims - 1]) cudaMemset(c->d_cells, 0, c->local_cells * 4);
    if (cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->ws_done, cudaEventDisableTiming) != cudaSuccess ||
        cudaMalloc(&c->d_counter, 4 * sizeof(unsigned long long)) != cudaSuccess ||
        cudaMemset(c->d_counter, 0, 4 * sizeof(unsigned long long)) != cudaSuccess ||
        cudaMalloc(&c->d_ctl, 64) != cudaSuccess || cudaMemset(c->d_ctl, 0, 64) != cudaSuccess) {
        rc = set_error(OLAP_E_CUDA, "stream/event/counter setup failed");
        olap_cube_destroy(c);
        return rc;
    }
    cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, device);
    int bps = 0;
    cudaFuncSetAttribute(reduce_kernel<int32_t, AccI>, cudaFuncAttributePreferredSharedMemoryCarveout,
                         cudaSharedmemCarveoutMaxL1);
    cudaFuncSetAttribute(reduce_kernel<float, AccF>, cudaFuncAttributePreferredSharedMemoryCarveout,
                         cudaSharedmemCarveoutMaxL1);
    // (no max-L1 carveout for reduce_kernel_w: its 2 KiB of per-warp descriptors would then
    // fit only 2 blocks per SM -- measured: C5 -40%)
    {
        int bw = 0;  // one grid serves both item kernels: the smaller residency of the two
        if (dtype == OLAP_INT32) {
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, reduce_kernel<int32_t, AccI>, kThreads, 0);
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bw, reduce_kernel_w<int32_t, AccI>, kThreads, 0);
        } else {
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, reduce_kernel<float, AccF>, kThreads, 0);
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bw, reduce_kernel_w<float, AccF>, kThreads, 0);
        }
        bps = std::min(bps, bw);
    }
    if (const char* s = getenv("OLAP_BLOCKS_PER_SM")) {
        int v = atoi(s);
        if (v > 0 && v < bps) bps = v;
    }
    c->blocks_per_sm = std::max(bps, 1);
    if (const char* s = getenv("OLAP_L2_FETCH")) cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, atoi(s));
    // L2-aware item order for cubes larger than 64 MiB: buckets of >= 8 MiB, <= kMaxBuckets of them
    if (c->local_cells * 4 > (64ll << 20) && !getenv("OLAP_NO_ORDER")) {
        int sh = 21;  // 2^21 cells = 8 MiB
        while ((c->local_cells >> sh) >= kMaxBuckets) ++sh;
        c->order_shift = sh;
    }
    c->d_ttot = reinterpret_cast<unsigned long long*>(c->d_ctl + 8);
    make_tiles(c);

    *out = c;
    return OLAP_OK;
}

int olap_cube_create_layout(int ndims, const int64_t* extents, int dtype, const olap_shard* shard, int device,
                            int layout, olap_cube** out) {
    clear_error();
    if (layout == OLAP_LAYOUT_ROWMAJOR) return olap_cube_create(ndims, extents, dtype, shard, device, out);
    if (layout != OLAP_LAYOUT_BRICK && layout != OLAP_LAYOUT_BRICK3)
        return set_error(OLAP_E_INVALID, "unknown layout %d", layout);
    if (!out || !extents) return set_error(OLAP_E_INVALID, "olap_cube_create_layout: NULL argument");
    if (ndims < 3 || ndims > kMaxDims - 2)
        return set_error(OLAP_E_INVALID, "bricked layout needs ndims in [3,%d], got %d", kMaxDims - 2, ndims);
    for (int k = 0; k < ndims; ++k)
        if (extents[k] < 1) return set_error(OLAP_E_INVALID, "extent[%d] = %lld < 1", k, (long long)extents[k]);
    olap_shard sh{1, 0, 1};
    if (shard) sh = *shard;
    if (sh.nshards < 1 || sh.shard < 0 || sh.shard >= sh.nshards || sh.block < 1)
        return set_error(OLAP_E_INVALID, "bad shard {%lld,%lld,%lld}", (long long)sh.nshards, (long long)sh.shard,
                         (long long)sh.block);
    const BrickDims bd = brick_dims(layout);
    // 2 x 4 x 4 bricks of a 3-D cube pair SHARD-LOCAL rows: the inner cube is this shard's own
    // (unsharded, ceil(local rows / 2) inner rows); otherwise dim 0 stays unbricked and the inner
    // cube is sharded like the logical one.
    const bool pair_rows = ndims == 3 && bd.a0 == 2;
    const int64_t lrows = shard_rows(extents[0], sh.nshards, sh.shard, sh.block);
    int64_t e[kMaxDims];
    for (int k = 0; k < ndims - 3; ++k) e[k] = extents[k];
    e[ndims - 3] = pair_rows ? std::max<int64_t>(1, (lrows + 1) / 2) : (extents[ndims - 3] + bd.a0 - 1) / bd.a0;
    e[ndims - 2] = (extents[ndims - 2] + bd.a - 1) / bd.a;
    e[ndims - 1] = (extents[ndims - 1] + bd.b - 1) / bd.b;
    e[ndims] = 32;
    olap_cube* ic = nullptr;
    int rc = olap_cube_create(ndims + 1, e, dtype, pair_rows ? nullptr : &sh, device, &ic);
    if (rc) return rc;
    if ((ic->local_cells >> 5) >= (1ll << 32)) {  // brick indices are 32-bit (2^32 bricks = 512 GiB per shard)
        olap_cube_destroy(ic);
        return set_error(OLAP_E_UNSUPPORTED, "a bricked shard must hold < 2^32 bricks");
    }
    // padding cells (ragged bricks, the unpaired last local row) read as 0 (they are always masked)
    if (cudaMemset(ic->d_cells, 0, ic->local_cells * 4) != cudaSuccess) {
        olap_cube_destroy(ic);
        return set_error(OLAP_E_CUDA, "cudaMemset of the brick array failed");
    }
    DeviceGuard dg(device);
    olap_cube* c = new (std::nothrow) olap_cube();
    if (!c) {
        olap_cube_destroy(ic);
        return set_error(OLAP_E_NOMEM, "host allocation failed");
    }
    ic->tiles_on = false;  // bricked queries run brick_reduce_kernel on the inner cube, never its tile path
    c->inner = ic;
    c->layout = layout;
    c->nd = ndims;
    c->dtype = dtype;
    c->device = device;
    c->sh = sh;
    for (int k = 0; k < ndims; ++k) c->n[k] = extents[k];
    c->pitch = c->n[ndims - 1];
    c->stride[ndims - 1] = 1;
    for (int k = ndims - 2; k >= 0; --k) c->stride[k] = c->stride[k + 1] * c->n[k + 1];
    c->lrow_cells = c->stride[0];
    c->row_cells = ic->row_cells;  // storage
    c->local_rows = lrows;
    c->local_cells = ic->local_cells;
    c->d_cells = ic->d_cells;
    c->num_sms = ic->num_sms;
    c->blocks_per_sm = ic->blocks_per_sm;
    if (cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->ws_done, cudaEventDisableTiming) != cudaSuccess) {
        rc = set_error(OLAP_E_CUDA, "stream/event setup failed");
        olap_cube_destroy(c);
        return rc;
    }
    *out = c;
    return OLAP_OK;
}

int olap_cube_info(const olap_cube* c, int64_t* local_rows, int64_t* local_cells, void** d_cells) {
    clear_error();
    if (!c) return set_error(OLAP_E_INVALID, "cube handle is NULL");
    if (c->multi()) {  // a group: every shard's rows and cells; no single device pointer
        int64_t r = 0, n = 0;
        for (const olap_cube* s : c->shards) {
            r += s->local_rows;
            n += s->local_cells;
        }
        if (local_rows) *local_rows = r;
        if (local_cells) *local_cells = n;
        if (d_cells) *d_cells = nullptr;
        return OLAP_OK;
    }
    if (local_rows) *local_rows = c->local_rows;
    if (local_cells) *local_cells = c->local_cells;
    if (d_cells) *d_cells = c->d_cells;
    return OLAP_OK;
}

int olap_cube_load_rows(olap_cube* c, int64_t row_lo, int64_t row_hi, const void* cells) {
    clear_error();
    int rc = check_cube(c);
    if (rc) return rc;
    if (!cells || row_lo < 0 || row_hi > c->n[0] || row_lo > row_hi)
        return set_error(OLAP_E_INVALID, "olap_cube_load_rows: bad rows [%lld,%lld)", (long long)row_lo,
                         (long long)row_hi);
    if (c->multi()) {  // every shard copies the rows it owns
        for (olap_cube* sc : c->shards) {
            rc = olap_cube_load_rows(sc, row_lo, row_hi, cells);
            if (rc) return rc;
        }
        return OLAP_OK;
    }
    std::lock_guard<std::mutex> lk(c->mu);
    DeviceGuard dg(c->device);
    OLAP_CUDA_TRY(cudaEventSynchronize(c->ws_done));
    if (c->inner) {
        OLAP_CUDA_TRY(cudaEventSynchronize(c->inner->ws_done));
        return load_rows_brick(c, row_lo, row_hi, cells);
    }
    const int64_t rb = c->row_cells * 4, lrb = c->lrow_cells * 4;  // device (padded) / host row bytes
    const int64_t nin = c->n[c->nd - 1];
    const bool padded = c->pitch != nin;
    const char* src = static_cast<const char*>(cells);
    char* dst = static_cast<char*>(c->d_cells);
    const int64_t G = c->sh.nshards, g = c->sh.shard, b = c->sh.block;
    int64_t r = row_lo;
    while (r < row_hi) {
        // run of consecutive owned rows starting at r (or skip the unowned ones)
        const int64_t blk_end = (r / b + 1) * b;
        const int64_t end = std::min(blk_end, row_hi);
        const int64_t stop = G == 1 ? row_hi : end;  // unsharded: the whole remainder is owned and contiguous
        if (G == 1 || (r / b) % G == g) {
            const int64_t lr = shard_local_of(r, G, b);
            if (!padded)
                OLAP_CUDA_TRY(cudaMemcpy(dst + lr * rb, src + (r - row_lo) * lrb, (stop - r) * rb,
                                         cudaMemcpyHostToDevice));
            else  // innermost rows of nin cells land on a pitch of c->pitch cells
                OLAP_CUDA_TRY(cudaMemcpy2D(dst + lr * rb, c->pitch * 4, src + (r - row_lo) * lrb, nin * 4, nin * 4,
                                           (stop - r) * (c->lrow_cells / nin), cudaMemcpyHostToDevice));
        }
        r = stop;
    }
    return OLAP_OK;
}

int olap_cube_load(olap_cube* c, const void* cells, int64_t ncells) {
    clear_error();
    int rc = check_cube(c);
    if (rc) return rc;
    if (ncells != c->n[0] * c->lrow_cells)
        return set_error(OLAP_E_INVALID, "olap_cube_load: ncells %lld != %lld", (long long)ncells,
                         (long long)(c->n[0] * c->lrow_cells));
    return olap_cube_load_rows(c, 0, c->n[0], cells);
}

int olap_cube_fill(olap_cube* c, int generator, uint64_t seed, const double* params) {
    clear_error();
    int rc = check_cube(c);
    if (rc) return rc;
    if (generator != OLAP_GEN_UNIFORM && generator != OLAP_GEN_AFFINE)
        return set_error(OLAP_E_INVALID, "unknown generator %d", generator);
    if (generator == OLAP_GEN_AFFINE && !params) return set_error(OLAP_E_INVALID, "affine generator needs params");
    if (c->multi()) {  // the generators are functions of the global index: every shard fills its own rows
        for (olap_cube* sc : c->shards) {
            rc = olap_cube_fill(sc, generator, seed, params);
            if (rc) return rc;
        }
        return OLAP_OK;
    }
    std::lock_guard<std::mutex> lk(c->mu);
    DeviceGuard dg(c->device);
    FillParams fp;
    std::memset(&fp, 0, sizeof(fp));
    if (params)
        for (int k = 0; k <= c->nd; ++k) fp.c[k] = params[k];
    const int grid = c->num_sms * 8;
    ++c->kernel_launches;
    if (c->inner) {
        const olap_cube* ic = c->inner;
        OLAP_CUDA_TRY(cudaEventSynchronize(ic->ws_done));
        const int nd = c->nd;
        const BrickDims bd = brick_dims(c->layout);
        const int64_t NW = ic->n[nd - 3], NX = ic->n[nd - 2], NZ = ic->n[nd - 1];
        int64_t P1 = 1;  // digits of dims 1..N-4 per dim-0 row
        for (int k = 1; k <= nd - 4; ++k) P1 *= c->n[k];
        if (c->dtype == OLAP_INT32)
            fill_brick_kernel<int32_t><<<grid, 256, 0, c->stream>>>(static_cast<int32_t*>(c->d_cells), make_geo(c),
                                                                    ic->local_cells, NW, NX, NZ, bd.a0, bd.a, bd.b, P1,
                                                                    generator, seed, fp);
        else
            fill_brick_kernel<float><<<grid, 256, 0, c->stream>>>(static_cast<float*>(c->d_cells), make_geo(c),
                                                                  ic->local_cells, NW, NX, NZ, bd.a0, bd.a, bd.b, P1,
                                                                  generator, seed, fp);
        OLAP_CUDA_TRY(cudaGetLastError());
        OLAP_CUDA_TRY(cudaStreamSynchronize(c->stream));
        return OLAP_OK;
    }
    if (c->dtype == OLAP_INT32)
        fill_kernel<int32_t><<<grid, 256, 0, c->stream>>>(static_cast<int32_t*>(c->d_cells), make_geo(c), c->row_cells,
                                                          generator, seed, fp);
    else
        fill_kernel<float><<<grid, 256, 0, c->stream>>>(static_cast<float*>(c->d_cells), make_geo(c), c->row_cells,
                                                        generator, seed, fp);
    OLAP_CUDA_TRY(cudaGetLastError());
    OLAP_CUDA_TRY(cudaStreamSynchronize(c->stream));
    return OLAP_OK;
}

int olap_cube_add_facts_device(olap_cube* c, int64_t nrows, const int32_t* d_ids, const void* d_values, void* stream) {
    clear_error();
    int rc = check_cube(c);
    if (rc) return rc;
    if (nrows < 0) return set_error(OLAP_E_INVALID, "nrows < 0");
    if (nrows == 0) return OLAP_OK;
    if (!d_ids) return set_error(OLAP_E_INVALID, "d_ids is NULL");
    if (c->inner) return set_error(OLAP_E_UNSUPPORTED, "olap_cube_add_facts_device needs a row-major cube");
    if (c->multi()) return set_error(OLAP_E_UNSUPPORTED, "olap_cube_add_facts_device: add facts to each shard");
    std::lock_guard<std::mutex> lk(c->mu);
    DeviceGuard dg(c->device);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    OLAP_CUDA_TRY(cudaStreamWaitEvent(st, c->ws_done, 0));
    const int grid = (int)std::min<int64_t>((nrows + 255) / 256, (int64_t)c->num_sms * 16);
    if (c->dtype == OLAP_INT32) {  // wraparound int32 adds are exact in any order: atomics
        ++c->kernel_launches;
        add_facts_kernel<int32_t><<<grid, 256, 0, st>>>(static_cast<int32_t*>(c->d_cells), make_geo(c), nrows, d_ids,
                                                        static_cast<const int32_t*>(d_values));
        OLAP_CUDA_TRY(cudaGetLastError());
    } else {
        // float32: sort the rows by cell (stable LSD radix sort, rows stay in order within a cell),
        // then add each cell's values in row order in fp64 and round once (fact_segsum_kernel)
        if (nrows > INT32_MAX) return set_error(OLAP_E_UNSUPPORTED, "a float32 build takes < 2^31 rows per call");
        int bits = 1;
        while (bits < 63 && (1ull << bits) <= (unsigned long long)c->local_cells + 1) ++bits;
        unsigned long long *k0 = nullptr, *k1 = nullptr;
        int32_t *r0 = nullptr, *r1 = nullptr;
        void* tmp = nullptr;
        size_t tb = 0;
        OLAP_CUDA_TRY(cub::DeviceRadixSort::SortPairs(nullptr, tb, k0, k1, r0, r1, (int)nrows, 0, bits, st));
        OLAP_CUDA_TRY(cudaMallocAsync(reinterpret_cast<void**>(&k0), sizeof(unsigned long long) * nrows, st));
        OLAP_CUDA_TRY(cudaMallocAsync(reinterpret_cast<void**>(&k1), sizeof(unsigned long long) * nrows, st));
        OLAP_CUDA_TRY(cudaMallocAsync(reinterpret_cast<void**>(&r0), sizeof(int32_t) * nrows, st));
        OLAP_CUDA_TRY(cudaMallocAsync(reinterpret_cast<void**>(&r1), sizeof(int32_t) * nrows, st));
        OLAP_CUDA_TRY(cudaMallocAsync(&tmp, std::max<size_t>(tb, 16), st));
        fact_cell_kernel<<<grid, 256, 0, st>>>(make_geo(c), nrows, d_ids, k0, r0);
        // keys < local_cells < 2^bits - 1: sorting the low `bits` bits puts kNoCell (all ones) last
        OLAP_CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp, tb, k0, k1, r0, r1, (int)nrows, 0, bits, st));
        fact_segsum_kernel<<<grid, 256, 0, st>>>(static_cast<float*>(c->d_cells), nrows, k1, r1,
                                                 static_cast<const float*>(d_values));
        OLAP_CUDA_TRY(cudaGetLastError());
        cudaFreeAsync(tmp, st);
        cudaFreeAsync(k0, st);
        cudaFreeAsync(k1, st);
        cudaFreeAsync(r0, st);
        cudaFreeAsync(r1, st);
        c->kernel_launches += 4;  // cells, radix sort (2 passes counted as one launch group), segment sums
    }
    OLAP_CUDA_TRY(cudaEventRecord(c->ws_done, st));
    return OLAP_OK;
}

int olap_cube_destroy(olap_cube* c) {
    clear_error();
    if (!c) return OLAP_OK;
    olap::exec_destroy(c->exec);  // drains its streams first
    c->exec = nullptr;
    if (c->multi()) {
        for (olap_cube* sc : c->shards) olap_cube_destroy(sc);
        delete c;
        return OLAP_OK;
    }
    DeviceGuard dg(c->device);
    if (c->ws_done) cudaEventSynchronize(c->ws_done);
    if (c->stream) cudaStreamSynchronize(c->stream);
    if (c->inner) {
        olap_cube_destroy(c->inner);
        c->inner = nullptr;
        c->d_cells = nullptr;  // owned by the inner cube
    }
    for (auto& g : c->graphs) cudaGraphExecDestroy(g.exec);
    c->graphs.clear();
    free_ws(c);
    cudaFree(c->d_ranges);
    cudaFree(c->d_ops);
    cudaFree(c->d_results);
    cudaFree(c->d_psum);
    cudaFree(c->d_pext);
    cudaFreeHost(c->h_pinned);
    cudaFree(c->d_counter);
    cudaFree(c->d_ctl);
    cudaFree(c->d_cells);
    for (auto e : c->ev) cudaEventDestroy(e);
    if (c->ws_done) cudaEventDestroy(c->ws_done);
    if (c->stream) cudaStreamDestroy(c->stream);
    delete c;
    return OLAP_OK;
}

int olap_query_batch(olap_cube* c, int64_t nq, const olap_range* ranges, const int32_t* ops, olap_result* results) {
    clear_error();
    int rc = check_cube(c);
    if (rc) return rc;
    if (nq < 0) return set_error(OLAP_E_INVALID, "nq < 0");
    if (nq == 0) return OLAP_OK;
    if (!ranges || !ops || !results) return set_error(OLAP_E_INVALID, "olap_query_batch: NULL buffer");
    rc = olap::validate_queries(c->nd, c->n, nq, ranges, ops);
    if (rc) return rc;
    if (c->multi() || c->comm) return olap::exec_query_batch(c->exec, nq, ranges, ops, results);
    if (c->sh.nshards != 1)
        return set_error(OLAP_E_STATE, "olap_query_batch on a shard needs an attached communicator "
                         "(olap_cube_attach_comm) or olap_query_partials_device");
    std::lock_guard<std::mutex> lk(c->mu);
    DeviceGuard dg(c->device);
    rc = ensure_stage(c, nq);
    if (rc) return rc;
    const size_t rbytes = sizeof(olap_range) * c->nd * nq, obytes = sizeof(int32_t) * nq,
                 res_bytes = sizeof(olap_result) * nq;
    char* hp = static_cast<char*>(c->h_pinned);
    OLAP_CUDA_TRY(cudaEventSynchronize(c->ws_done));  // pinned staging reuse
    std::memcpy(hp, ranges, rbytes);
    std::memcpy(hp + rbytes, ops, obytes);
    cudaStream_t st = c->stream;
    char* hres = hp + rbytes + obytes;
    auto enqueue = [&]() -> int {
        OLAP_CUDA_TRY(cudaMemcpyAsync(c->d_ranges, hp, rbytes, cudaMemcpyHostToDevice, st));
        OLAP_CUDA_TRY(cudaMemcpyAsync(c->d_ops, hp + rbytes, obytes, cudaMemcpyHostToDevice, st));
        int r = run_partials(c, nq, c->d_ranges, c->d_ops, c->d_psum, c->d_pext, st);
        if (r) return r;
        r = launch_finalize(c->nd, c->n, c->dtype, nq, c->d_ranges, c->d_ops, c->d_psum, c->d_pext, c->d_results,
                            st);
        if (r) return r;
        OLAP_CUDA_TRY(cudaMemcpyAsync(hres, c->d_results, res_bytes, cudaMemcpyDeviceToHost, st));
        return OLAP_OK;
    };
    // small batches: replay the batch's CUDA graph (launch-bound otherwise); not while
    // the reduce kernel is being timed (olap_cube_profile), whose events a graph does not record
    const bool graph = nq <= kGraphMaxQueries && !c->prof && !(c->inner && c->inner->prof) && !getenv("OLAP_NO_GRAPHS");
    if (graph) {
        olap_cube* wc = c->inner ? c->inner : c;
        rc = ensure_ws(wc, nq);  // the workspace cannot grow inside a capture
        if (rc) return rc;
        olap_cube::BatchGraph* g = nullptr;
        for (auto& e : c->graphs)
            if (e.nq == nq && e.gen == c->ws_gen + wc->ws_gen * 1000003ull) g = &e;
        if (!g) {
            if (c->graphs.size() >= 4) {  // evict the least recently used
                auto lru = std::min_element(c->graphs.begin(), c->graphs.end(),
                                            [](const auto& a, const auto& b) { return a.last < b.last; });
                cudaGraphExecDestroy(lru->exec);
                c->graphs.erase(lru);
            }
            const int64_t k0 = c->kernel_launches + (c->inner ? c->inner->kernel_launches : 0);
            const int64_t f0 = g_finalize_launches.load();
            OLAP_CUDA_TRY(cudaEventSynchronize(wc->ws_done));
            OLAP_CUDA_TRY(cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal));
            rc = enqueue();
            cudaGraph_t gr = nullptr;
            const cudaError_t ce = cudaStreamEndCapture(st, &gr);
            if (rc) {
                if (gr) cudaGraphDestroy(gr);
                return rc;
            }
            OLAP_CUDA_TRY(ce);
            olap_cube::BatchGraph ng;
            ng.nq = nq;
            ng.gen = c->ws_gen + wc->ws_gen * 1000003ull;
            ng.kernels = c->kernel_launches + (c->inner ? c->inner->kernel_launches : 0) - k0;
            ng.finals = g_finalize_launches.load() - f0;
            const cudaError_t ie = cudaGraphInstantiate(&ng.exec, gr, 0);
            cudaGraphDestroy(gr);
            OLAP_CUDA_TRY(ie);
            c->graphs.push_back(ng);
            g = &c->graphs.back();
        } else {  // the kernels a replay launches count like launched ones (olap_cube_stats)
            c->kernel_launches += g->kernels;
            g_finalize_launches.fetch_add(g->finals);
        }
        g->last = ++c->graph_clock;
        OLAP_CUDA_TRY(cudaStreamWaitEvent(st, wc->ws_done, 0));  // a device batch on another stream
        OLAP_CUDA_TRY(cudaGraphLaunch(g->exec, st));
        if (c->inner) OLAP_CUDA_TRY(cudaEventRecord(c->inner->ws_done, st));
    } else {
        rc = enqueue();
        if (rc) return rc;
    }
    OLAP_CUDA_TRY(cudaEventRecord(c->ws_done, st));
    OLAP_CUDA_TRY(cudaStreamSynchronize(st));
    std::memcpy(results, hres, res_bytes);
    return OLAP_OK;
}

int olap_query_partials_device(olap_cube* c, int64_t nq, const olap_range* d_ranges, const int32_t* d_ops,
                               int64_t* d_sum, int32_t* d_ext, void* stream) {
    clear_error();
    int rc = check_cube(c);
    if (rc) return rc;
    if (nq < 0) return set_error(OLAP_E_INVALID, "nq < 0");
    if (nq == 0) return OLAP_OK;
    if (!d_ranges || !d_ops || !d_sum || !d_ext) return set_error(OLAP_E_INVALID, "NULL device buffer");
    if (c->multi())
        return set_error(OLAP_E_UNSUPPORTED, "olap_query_partials_device on a group handle: query its shards, or use "
                         "olap_query_batch(_device)");
    std::lock_guard<std::mutex> lk(c->mu);
    DeviceGuard dg(c->device);
    return run_partials(c, nq, d_ranges, d_ops, d_sum, d_ext, static_cast<cudaStream_t>(stream));
}

int olap_query_batch_device(olap_cube* c, int64_t nq, const olap_range* d_ranges, const int32_t* d_ops,
                            olap_result* d_results, void* stream) {
    clear_error();
    int rc = check_cube(c);
    if (rc) return rc;
    if (nq < 0) return set_error(OLAP_E_INVALID, "nq < 0");
    if (nq == 0) return OLAP_OK;
    if (!d_ranges || !d_ops || !d_results) return set_error(OLAP_E_INVALID, "NULL device buffer");
    if (c->multi() || c->comm) {
        if (capturing(static_cast<cudaStream_t>(stream)))
            return set_error(OLAP_E_UNSUPPORTED, "stream capture of a multi-GPU batch");
        return olap::exec_query_batch_device(c->exec, nq, d_ranges, d_ops, d_results, static_cast<cudaStream_t>(stream));
    }
    if (c->sh.nshards != 1)
        return set_error(OLAP_E_STATE, "olap_query_batch_device on a shard needs an attached communicator");
    std::lock_guard<std::mutex> lk(c->mu);
    DeviceGuard dg(c->device);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    const bool cap = capturing(st);
    if (cap && nq > c->stage_cap)
        return set_error(OLAP_E_STATE, "stream capture: run one batch of %lld queries outside capture first",
                         (long long)nq);
    rc = ensure_stage(c, nq);
    if (rc) return rc;
    rc = run_partials(c, nq, d_ranges, d_ops, c->d_psum, c->d_pext, st);
    if (rc) return rc;
    rc = launch_finalize(c->nd, c->n, c->dtype, nq, d_ranges, d_ops, c->d_psum, c->d_pext, d_results, st);
    if (rc) return rc;
    if (!cap) OLAP_CUDA_TRY(cudaEventRecord(c->ws_done, st));
    return OLAP_OK;
}

int olap_partials_combine_device(int dtype, int64_t nq, const int64_t* d_sum_in, const int32_t* d_ext_in,
                                 int64_t* d_sum_acc, int32_t* d_ext_acc, void* stream) {
    clear_error();
    if (dtype != OLAP_INT32 && dtype != OLAP_FLOAT32) return set_error(OLAP_E_INVALID, "bad dtype %d", dtype);
    if (nq < 0) return set_error(OLAP_E_INVALID, "nq < 0");
    if (nq == 0) return OLAP_OK;
    if (!d_sum_in || !d_ext_in || !d_sum_acc || !d_ext_acc) return set_error(OLAP_E_INVALID, "NULL device buffer");
    const int grid = (int)std::min<int64_t>((nq + 255) / 256, 4096);
    combine_kernel<<<grid, 256, 0, static_cast<cudaStream_t>(stream)>>>(dtype, nq, d_sum_in, d_ext_in, d_sum_acc,
                                                                         d_ext_acc);
    OLAP_CUDA_TRY(cudaGetLastError());
    return OLAP_OK;
}

int olap_finalize_device(int ndims, const int64_t* extents, int dtype, int64_t nq, const olap_range* d_ranges,
                         const int32_t* d_ops, const int64_t* d_sum, const int32_t* d_ext, olap_result* d_results,
                         void* stream) {
    clear_error();
    if (ndims < 1 || ndims > kMaxDims || !extents) return set_error(OLAP_E_INVALID, "bad ndims/extents");
    if (dtype != OLAP_INT32 && dtype != OLAP_FLOAT32) return set_error(OLAP_E_INVALID, "bad dtype %d", dtype);
    if (nq < 0) return set_error(OLAP_E_INVALID, "nq < 0");
    if (nq == 0) return OLAP_OK;
    if (!d_ranges || !d_ops || !d_sum || !d_ext || !d_results) return set_error(OLAP_E_INVALID, "NULL device buffer");
    return launch_finalize(ndims, extents, dtype, nq, d_ranges, d_ops, d_sum, d_ext, d_results,
                           static_cast<cudaStream_t>(stream));
}

int olap_shard_local_rows(int64_t n0, const olap_shard* s, int64_t lo, int64_t hi, int64_t* llo, int64_t* lhi) {
    clear_error();
    if (!llo || !lhi || n0 < 1) return set_error(OLAP_E_INVALID, "olap_shard_local_rows: bad argument");
    olap_shard sh{1, 0, 1};
    if (s) sh = *s;
    if (sh.nshards < 1 || sh.shard < 0 || sh.shard >= sh.nshards || sh.block < 1)
        return set_error(OLAP_E_INVALID, "bad shard");
    if (lo < 0 || hi >= n0) return set_error(OLAP_E_RANGE, "rows [%lld,%lld] outside [0,%lld)", (long long)lo,
                                             (long long)hi, (long long)n0);
    int64_t a = 1, b = 0;
    if (lo <= hi && shard_local_range(n0, sh.nshards, sh.shard, sh.block, lo, hi, &a, &b)) {
        *llo = a;
        *lhi = b;
    } else {
        *llo = 1;
        *lhi = 0;
    }
    return OLAP_OK;
}

int olap_cube_stats(const olap_cube* c, int64_t* kernel_launches, int* l2_order) {
    clear_error();
    if (!c) return set_error(OLAP_E_INVALID, "cube handle is NULL");
    if (c->multi()) {
        int64_t k = olap::exec_launches(c->exec);
        int o = 1;
        for (const olap_cube* sc : c->shards) {
            int64_t ks = 0;
            int os = 0;
            olap_cube_stats(sc, &ks, &os);
            k += ks;
            o &= os;
        }
        if (kernel_launches) *kernel_launches = k;
        if (l2_order) *l2_order = o;
        return OLAP_OK;
    }
    const olap_cube* ic = c->inner ? c->inner : c;
    if (kernel_launches)
        *kernel_launches = c->kernel_launches + (c->inner ? c->inner->kernel_launches : 0) + olap::exec_launches(c->exec);
    if (l2_order) *l2_order = ic->order_shift >= 0 ? 1 : 0;
    return OLAP_OK;
}

int64_t olap_finalize_launches(void) { return g_finalize_launches.load(); }

int olap_cube_tile_stats(olap_cube* c, int* enabled, int64_t* tile_cells, int64_t* ntiles, int* last_used) {
    clear_error();
    if (!c) return set_error(OLAP_E_INVALID, "cube handle is NULL");
    if (c->multi()) return olap_cube_tile_stats(c->shards[0], enabled, tile_cells, ntiles, last_used);
    if (c->inner) {
        std::lock_guard<std::mutex> lk(c->mu);
        return olap_cube_tile_stats(c->inner, enabled, tile_cells, ntiles, last_used);
    }
    std::lock_guard<std::mutex> lk(c->mu);
    DeviceGuard dg(c->device);
    OLAP_CUDA_TRY(cudaEventSynchronize(c->ws_done));
    int32_t mode = 0;
    OLAP_CUDA_TRY(cudaMemcpy(&mode, c->d_ctl, sizeof(mode), cudaMemcpyDeviceToHost));
    if (enabled) *enabled = c->tiles_on ? 1 : 0;
    if (tile_cells) *tile_cells = c->tg.tcells;
    if (ntiles) *ntiles = c->tg.ntiles;
    if (last_used) *last_used = mode;
    return OLAP_OK;
}

int olap_cube_profile(olap_cube* c, int enable) {
    clear_error();
    if (!c) return set_error(OLAP_E_INVALID, "cube handle is NULL");
    if (c->multi()) {
        for (olap_cube* sc : c->shards) {
            int rc = olap_cube_profile(sc, enable);
            if (rc) return rc;
        }
        return OLAP_OK;
    }
    if (c->inner) {
        std::lock_guard<std::mutex> lk(c->mu);
        return olap_cube_profile(c->inner, enable);
    }
    std::lock_guard<std::mutex> lk(c->mu);
    DeviceGuard dg(c->device);
    OLAP_CUDA_TRY(cudaEventSynchronize(c->ws_done));
    c->prof = enable != 0;
    c->ev_used = 0;
    c->launches = 0;
    OLAP_CUDA_TRY(cudaMemcpy(&c->bytes_base, c->d_counter + 1, sizeof(unsigned long long), cudaMemcpyDeviceToHost));
    return OLAP_OK;
}

int olap_cube_profile_read(olap_cube* c, double* reduce_ms, int64_t* launches, int64_t* bytes) {
    clear_error();
    if (!c) return set_error(OLAP_E_INVALID, "cube handle is NULL");
    if (c->multi()) {  // sums over the shards (reduce time: summed over shards, whatever device)
        double ms = 0.0;
        int64_t n = 0, b = 0;
        for (olap_cube* sc : c->shards) {
            double m = 0.0;
            int64_t nn = 0, bb = 0;
            int rc = olap_cube_profile_read(sc, &m, &nn, &bb);
            if (rc) return rc;
            ms += m;
            n += nn;
            b += bb;
        }
        if (reduce_ms) *reduce_ms = ms;
        if (launches) *launches = n;
        if (bytes) *bytes = b;
        return OLAP_OK;
    }
    if (c->inner) {
        std::lock_guard<std::mutex> lk(c->mu);
        OLAP_CUDA_TRY(cudaEventSynchronize(c->ws_done));
        return olap_cube_profile_read(c->inner, reduce_ms, launches, bytes);
    }
    std::lock_guard<std::mutex> lk(c->mu);
    DeviceGuard dg(c->device);
    OLAP_CUDA_TRY(cudaEventSynchronize(c->ws_done));
    double ms = 0.0;
    for (size_t i = 0; i + 1 < c->ev_used; i += 2) {
        float t = 0.f;
        OLAP_CUDA_TRY(cudaEventSynchronize(c->ev[i + 1]));
        OLAP_CUDA_TRY(cudaEventElapsedTime(&t, c->ev[i], c->ev[i + 1]));
        ms += t;
    }
    unsigned long long b = 0;
    OLAP_CUDA_TRY(cudaMemcpy(&b, c->d_counter + 1, sizeof(b), cudaMemcpyDeviceToHost));
    if (reduce_ms) *reduce_ms = ms;
    if (launches) *launches = c->launches;
    if (bytes) *bytes = (int64_t)(b - c->bytes_base);
    return OLAP_OK;
}

int olap_cube_create_multi(int ndims, const int64_t* extents, int dtype, const olap_cube_opts* opts, olap_cube** out) {
    clear_error();
    if (!out || !extents || !opts || !opts->devices)
        return set_error(OLAP_E_INVALID, "olap_cube_create_multi: NULL argument");
    if (opts->ndevices < 1 || opts->ndevices > 64)
        return set_error(OLAP_E_INVALID, "ndevices %d not in [1,64]", opts->ndevices);
    if (opts->shards_per_device < 1 || opts->shard_block < 1)
        return set_error(OLAP_E_INVALID, "shards_per_device and shard_block must be >= 1");
    if (ndims < 1 || ndims > kMaxDims) return set_error(OLAP_E_INVALID, "ndims %d not in [1,8]", ndims);
    for (int i = 0; i < opts->ndevices; ++i)
        for (int j = 0; j < i; ++j)
            if (opts->devices[i] == opts->devices[j])
                return set_error(OLAP_E_INVALID, "device %d listed twice (use shards_per_device)", opts->devices[i]);
    const int spd = opts->shards_per_device;
    const int64_t G = (int64_t)opts->ndevices * spd;
    olap_cube* c = new (std::nothrow) olap_cube();
    if (!c) return set_error(OLAP_E_NOMEM, "host allocation failed");
    c->nd = ndims;
    c->dtype = dtype;
    c->device = opts->devices[0];
    c->sh = olap_shard{G, 0, opts->shard_block};
    for (int k = 0; k < ndims; ++k) c->n[k] = extents[k];
    c->lrow_cells = 1;
    for (int k = 1; k < ndims; ++k) c->lrow_cells *= extents[k];
    olap::ExecSpec spec;
    spec.nd = ndims;
    spec.dtype = dtype;
    for (int k = 0; k < ndims; ++k) spec.n[k] = extents[k];
    spec.spd = spd;
    spec.own_comms = true;
    for (int i = 0; i < opts->ndevices; ++i) spec.devices.push_back(opts->devices[i]);
    for (int64_t g = 0; g < G; ++g) {
        const olap_shard sh{G, g, opts->shard_block};
        olap_cube* sc = nullptr;
        int rc = olap_cube_create_layout(ndims, extents, dtype, &sh, opts->devices[g / spd], opts->layout, &sc);
        if (rc) {
            std::string msg = olap_last_error();
            olap_cube_destroy(c);
            return set_error(rc, "shard %lld of %lld on device %d: %s", (long long)g, (long long)G,
                             opts->devices[g / spd], msg.c_str());
        }
        c->shards.push_back(sc);
    }
    spec.shards = c->shards;
    int rc = olap::exec_create(spec, &c->exec);
    if (rc) {
        std::string msg = olap_last_error();
        olap_cube_destroy(c);
        return set_error(rc, "%s", msg.c_str());
    }
    *out = c;
    return OLAP_OK;
}

int olap_cube_attach_comm(olap_cube* c, olap_comm* comm) {
    clear_error();
    int rc = check_cube(c);
    if (rc) return rc;
    if (c->multi()) return set_error(OLAP_E_INVALID, "a group handle has its own communicators");
    int nranks = 0, rank = 0, device = 0;
    if (comm) {
        rc = olap_comm_info(comm, &nranks, &rank, &device);
        if (rc) return rc;
        if (c->sh.nshards != nranks || c->sh.shard != rank || c->device != device)
            return set_error(OLAP_E_INVALID, "cube shard %lld of %lld on device %d does not match communicator rank %d "
                             "of %d on device %d", (long long)c->sh.shard, (long long)c->sh.nshards, c->device, rank,
                             nranks, device);
    }
    olap::exec_destroy(c->exec);
    c->exec = nullptr;
    c->comm = nullptr;
    if (!comm) return OLAP_OK;
    olap::ExecSpec spec;
    spec.nd = c->nd;
    spec.dtype = c->dtype;
    for (int k = 0; k < c->nd; ++k) spec.n[k] = c->n[k];
    spec.devices.push_back(c->device);
    spec.shards.push_back(c);
    spec.comm = comm;
    rc = olap::exec_create(spec, &c->exec);
    if (rc) return rc;
    c->comm = comm;
    return OLAP_OK;
}

int olap_query_stream(olap_cube* c, int64_t nq, const olap_range* ranges, const int32_t* ops, olap_result* results,
                      int64_t batch) {
    clear_error();
    int rc = check_cube(c);
    if (rc) return rc;
    if (nq < 0) return set_error(OLAP_E_INVALID, "nq < 0");
    if (nq == 0) return OLAP_OK;
    if (!ranges || !ops || !results) return set_error(OLAP_E_INVALID, "olap_query_stream: NULL buffer");
    rc = olap::validate_queries(c->nd, c->n, nq, ranges, ops);
    if (rc) return rc;
    if (!c->exec) {
        if (c->sh.nshards != 1)
            return set_error(OLAP_E_STATE, "olap_query_stream on a shard needs an attached communicator");
        olap::ExecSpec spec;  // a plain cube: the pipeline without an exchange
        spec.nd = c->nd;
        spec.dtype = c->dtype;
        for (int k = 0; k < c->nd; ++k) spec.n[k] = c->n[k];
        spec.devices.push_back(c->device);
        spec.shards.push_back(c);
        rc = olap::exec_create(spec, &c->exec);
        if (rc) return rc;
    }
    return olap::exec_query_stream(c->exec, nq, ranges, ops, results, batch);
}

}  // extern "C"
