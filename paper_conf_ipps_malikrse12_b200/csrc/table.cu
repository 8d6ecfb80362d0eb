// table.cu — the paper's own GPU path: queries Q_D (Eq. 11,
// PAPER.md:210-216) over a column-store fact table held in GPU memory ("a 1D array
// memory structure ... placing all columns of the table one after another",
// PAPER.md:206).  A query is a set of conditions C_L(f, t, l_K) — one column (dimension
// L at level K) and an inclusive id range — plus a data column and an aggregate op; a
// row contributes when it satisfies every condition.
//
// The paper ran one query per SM partition and read each referenced column whole per
// query (Eq. 12: bytes = rows x C_QD x 4).  B200 design: a SHARED scan — one persistent
// launch per batch streams every column once, tile by tile, into shared memory, and
// every warp evaluates its share of the batch's queries on the staged tile (each
// condition one unsigned range compare).  Per-(tile range, query) partials are folded in
// fixed range order by a second kernel, so results are deterministic.
#include <algorithm>
#include <climits>
#include <cstring>
#include <mutex>
#include <new>
#include <vector>

#include "common.cuh"

namespace olap {

constexpr int kMaxTableCols = 16;
constexpr int kMaxConds = 16;
constexpr int kTileRows = 1024;
#ifndef OLAP_SPARSE_ROWS
#define OLAP_SPARSE_ROWS 6
#endif
constexpr int kSparseRows = OLAP_SPARSE_ROWS;  // a lane with <= this many surviving rows checks them one by one
constexpr int kScanWarps = 8;
constexpr int kScanThreads = kScanWarps * 32;

// Condition in the kernel's form: row value v passes iff (uint32)(v - lo) <= span.
struct TCond {
    int32_t col;
    uint32_t lo;
    uint32_t span;
};

struct TQuery {
    int32_t ncond;
    int32_t data_col;
    int32_t op;
    int32_t flags;  // OLAP_RESULT_INVALID / impossible (some condition empty)
    TCond c[kMaxConds];
};

struct TPartial {  // per (tile range, query)
    long long sum;     // int64 wraparound sum or double bits
    int64_t count;     // matching rows
    int32_t code_max;  // order-preserving code of MAX (INT_MIN = none)
    int32_t code_min;  // ~code of MIN           (INT_MIN = none)
};

struct TableCols {
    const uint32_t* col[kMaxTableCols];
    int32_t dtype[kMaxTableCols];
};

__device__ __forceinline__ int32_t tf32_code(float f) {
    const int32_t b = __float_as_int(f);
    return b ^ ((b >> 31) & 0x7fffffff);
}
__device__ __forceinline__ float tf32_decode(int32_t c) { return __int_as_float(c ^ ((c >> 31) & 0x7fffffff)); }

// Columns the batch reads (Eq. 12): every condition's column, and the
// data column unless the query is COUNT.  A query that cannot match reads nothing.
// Called by every thread of a query-per-thread kernel (the trailing threads of the last
// block return early, so the OR is a plain atomic, not a warp-collective one).
__device__ __forceinline__ void note_columns(const TQuery& t, uint32_t* colmask) {
    if (t.flags || t.ncond < 0) return;
    uint32_t m = t.op != OLAP_COUNT ? 1u << t.data_col : 0u;
    for (int k = 0; k < t.ncond; ++k) m |= 1u << t.c[k].col;
    if (m) atomicOr(colmask, m);
}

// Conditions in ascending span order (equality predicates first): after the most selective
// one, few rows of a lane survive and scan_query_tile checks the rest row by row.
__device__ __forceinline__ void order_conds(TQuery& t) {
    for (int i = 1; i < t.ncond; ++i) {
        const TCond x = t.c[i];
        int j = i - 1;
        while (j >= 0 && t.c[j].span > x.span) {
            t.c[j + 1] = t.c[j];
            --j;
        }
        t.c[j + 1] = x;
    }
}

// conditions -> TQuery (one thread per query)
__global__ void table_prep_kernel(int64_t nq, int ncols, TableCols tc, const int64_t* __restrict__ off,
                                  const olap_cond* __restrict__ conds, const int32_t* __restrict__ data_cols,
                                  const int32_t* __restrict__ ops, TQuery* __restrict__ qs,
                                  uint32_t* __restrict__ colmask) {
    const int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (q >= nq) return;
    TQuery t;
    t.flags = 0;
    t.op = ops[q];
    t.data_col = data_cols[q];
    const int64_t a = off[q], b = off[q + 1];
    t.ncond = (int32_t)(b - a);
    if (t.op < OLAP_SUM || t.op > OLAP_AVG || t.data_col < 0 || t.data_col >= ncols || b < a || b - a > kMaxConds)
        t.flags = OLAP_RESULT_INVALID;
    bool impossible = false;
    for (int64_t k = a; k < b && !t.flags; ++k) {
        const olap_cond c = conds[k];
        if (c.col < 0 || c.col >= ncols || tc.dtype[c.col] != OLAP_INT32) {
            t.flags = OLAP_RESULT_INVALID;
            break;
        }
        const int64_t lo = c.lo < INT_MIN ? (int64_t)INT_MIN : c.lo;
        const int64_t hi = c.hi > INT_MAX ? (int64_t)INT_MAX : c.hi;
        TCond& d = t.c[k - a];
        d.col = c.col;
        if (lo > hi) {
            impossible = true;
            d.lo = 0;
            d.span = 0;
        } else {
            d.lo = (uint32_t)(int32_t)lo;
            d.span = (uint32_t)(hi - lo);
        }
    }
    if (impossible && !t.flags) t.ncond = -1;  // no row can match
    if (!t.flags) order_conds(t);
    qs[q] = t;
    note_columns(t, colmask);
}

// Column-map of box queries: dimension d is column col[d] with members [0, extent[d]).
struct BoxMap {
    int32_t ndims;
    int32_t col[kMaxConds];
    int64_t extent[kMaxConds];
};

// boxes -> TQuery: a range covering the whole dimension is no condition (reads no column).
__global__ void table_prep_boxes_kernel(int64_t nq, int ncols, TableCols tc, BoxMap bm,
                                        const olap_range* __restrict__ boxes, const int32_t* __restrict__ data_cols,
                                        const int32_t* __restrict__ ops, TQuery* __restrict__ qs,
                                        uint32_t* __restrict__ colmask) {
    const int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (q >= nq) return;
    TQuery t;
    t.flags = 0;
    t.op = ops[q];
    t.data_col = data_cols[q];
    t.ncond = 0;
    if (t.op < OLAP_SUM || t.op > OLAP_AVG || t.data_col < 0 || t.data_col >= ncols) t.flags = OLAP_RESULT_INVALID;
    bool impossible = false;
    for (int d = 0; d < bm.ndims && !t.flags; ++d) {
        const olap_range r = boxes[q * bm.ndims + d];
        if (r.lo < 0 || r.hi >= bm.extent[d]) {  // outside [0, extent): INVALID, the cube path's rule (R10)
            t.flags = OLAP_RESULT_INVALID;
            break;
        }
        if (r.lo > r.hi) {
            impossible = true;
            continue;
        }
        if (r.lo <= 0 && r.hi >= bm.extent[d] - 1) continue;  // the whole dimension: no condition
        // ids are in [0, extent) (< 2^31 by the 32-bit id columns): clamp, then the span cannot wrap
        const int64_t lo = r.lo < INT_MIN ? (int64_t)INT_MIN : (r.lo > INT_MAX ? (int64_t)INT_MAX : r.lo);
        const int64_t hi = r.hi > INT_MAX ? (int64_t)INT_MAX : (r.hi < INT_MIN ? (int64_t)INT_MIN : r.hi);
        if (lo > hi) {
            impossible = true;
            continue;
        }
        TCond& c = t.c[t.ncond++];
        c.col = bm.col[d];
        c.lo = (uint32_t)(int32_t)lo;
        c.span = (uint32_t)(hi - lo);
    }
    if (impossible && !t.flags) t.ncond = -1;
    if (!t.flags) order_conds(t);
    qs[q] = t;
    note_columns(t, colmask);
}

// A query in the scan's shared-memory form (48 B, three broadcast LDS.128): the header, then its
// first kInlineConds conditions (ascending span); further conditions are read from its TQuery.
constexpr int kInlineConds = 4;
struct SQ {
    int32_t ncond;     // < 0: the query reads nothing (invalid or impossible)
    int32_t q;         // query index (TQuery of conditions beyond kInlineConds; partial slot)
    int32_t meta;      // data_col | fl << 8 (float data) | opk << 9 (0 SUM / AVG, 1 MIN, 2 MAX, 3 COUNT)
    uint32_t colpack;  // column of inline condition k in bits 4k .. 4k+3
    uint32_t lo[kInlineConds];
    uint32_t span[kInlineConds];
};
static_assert(sizeof(SQ) == 48, "three 16-B words per query");

// One query on one staged tile.  Lane l owns the row quads 4l..4l+3 + 128 i (i < 8): every
// condition column is read with one LDS.128 per quad (lane-consecutive 16-B chunks, no bank
// conflicts) and evaluated into a 32-bit pass mask (bit 4i + j = row 128 i + 4 l + j);
// COUNT is a popcount, and only matching rows touch the data column, folding only the
// accumulator the op needs (OPK: 0 SUM / AVG, 1 MIN, 2 MAX, 3 COUNT).  Returns false when no
// row of the tile matches (s, cnt, cmx, cmn untouched); else every lane holds the warp's totals.
__device__ __forceinline__ uint32_t quad_pass(uint4 x, uint32_t lo, uint32_t span) {
    return (uint32_t)(x.x - lo <= span) | (uint32_t)(x.y - lo <= span) << 1 | (uint32_t)(x.z - lo <= span) << 2 |
           (uint32_t)(x.w - lo <= span) << 3;
}
template <bool FLOAT_DATA, int OPK>
__device__ __forceinline__ bool scan_query_tile(const uint32_t* __restrict__ smem, int rows, const SQ* sq,
                                                const TQuery* __restrict__ qs, int lane, long long& s, int32_t& cnt,
                                                int32_t& cmx, int32_t& cmn) {
    static_assert(kTileRows == 1024, "one 32-bit pass mask per lane");
    uint32_t pass = rows >= kTileRows ? 0xFFFFFFFFu : 0u;
    if (rows < kTileRows)
        for (int b = 0; b < 32; ++b)
            if (128 * (b >> 2) + 4 * lane + (b & 3) < rows) pass |= 1u << b;
    const int nc = sq->ncond;
    for (int k = 0; k < nc && pass; ++k) {
        uint32_t col, lo, span;
        if (k < kInlineConds) {  // shared memory (broadcast)
            col = (sq->colpack >> (4 * k)) & 15u;
            lo = sq->lo[k];
            span = sq->span[k];
        } else {
            const TCond c = qs[sq->q].c[k];
            col = (uint32_t)c.col;
            lo = c.lo;
            span = c.span;
        }
        if (__popc(pass) <= kSparseRows) {  // few survivors: check them one by one
            const uint32_t* cp = smem + col * kTileRows + 4 * lane;
            uint32_t left = pass;
            while (left) {
                const int b = __ffs(left) - 1;
                left &= left - 1;
                if (cp[128 * (b >> 2) + (b & 3)] - lo > span) pass &= ~(1u << b);
            }
            continue;
        }
        const uint4* cp = reinterpret_cast<const uint4*>(smem + col * kTileRows) + lane;
        uint32_t m = 0;
#pragma unroll
        for (int i = 0; i < 8; ++i) m |= quad_pass(cp[32 * i], lo, span) << (4 * i);
        pass &= m;
    }
    // no row of the tile matches (most tiles of a query with equality predicates)
    if (!__any_sync(0xffffffffu, pass)) return false;
    int32_t n = __popc(pass);
    const uint32_t* data = smem + (sq->meta & 0xff) * kTileRows + 4 * lane;
    unsigned long long si = 0ull;
    double sf = 0.0;
    float fmn = __int_as_float(0x7f800000), fmx = __int_as_float(0xff800000);
    int32_t imn = INT_MAX, imx = INT_MIN;
    uint32_t bits_left = OPK == 3 ? 0u : pass;
    while (bits_left) {
        const int b = __ffs(bits_left) - 1;
        bits_left &= bits_left - 1;
        const uint32_t bits = data[128 * (b >> 2) + (b & 3)];
        if (FLOAT_DATA) {
            const float v = __uint_as_float(bits);
            if (OPK == 0) sf += (double)v;
            if (OPK == 1) fmn = fminf(fmn, v);
            if (OPK == 2) fmx = fmaxf(fmx, v);
        } else {
            const int32_t v = (int32_t)bits;
            if (OPK == 0) si += (unsigned long long)(long long)v;
            if (OPK == 1) imn = min(imn, v);
            if (OPK == 2) imx = max(imx, v);
        }
    }
    // warp reduction in fixed order (only the op's accumulator)
    if (OPK == 0) {
        long long sb = FLOAT_DATA ? __double_as_longlong(sf) : (long long)si;
#pragma unroll
        for (int o = 16; o; o >>= 1) {
            const long long so = __shfl_xor_sync(0xffffffffu, sb, o);
            sb = FLOAT_DATA ? __double_as_longlong(__longlong_as_double(sb) + __longlong_as_double(so))
                            : (long long)((unsigned long long)sb + (unsigned long long)so);
        }
        s = sb;
    }
    cnt = __reduce_add_sync(0xffffffffu, (uint32_t)n);
    if (OPK == 2) cmx = __reduce_max_sync(0xffffffffu, n ? (FLOAT_DATA ? tf32_code(fmx) : imx) : INT_MIN);
    if (OPK == 1) cmn = __reduce_max_sync(0xffffffffu, n ? ~(FLOAT_DATA ? tf32_code(fmn) : imn) : INT_MIN);
    return true;
}

// Scan instantiation of a query: (float data, op) -> 0..7; 8 = skipped (invalid / empty).
__device__ __forceinline__ int scan_class(const TableCols& tc, const TQuery& tq) {
    if (tq.flags || tq.ncond < 0) return 8;
    const int opk = tq.op == OLAP_MIN ? 1 : tq.op == OLAP_MAX ? 2 : tq.op == OLAP_COUNT ? 3 : 0;
    return (tc.dtype[tq.data_col] == OLAP_FLOAT32 ? 4 : 0) + opk;
}

// Batch order for the scan, grouped by scan_class: the warps of a block (and the blocks
// of the grid) then run the same scan_query_tile instantiation at the same time instead of
// cycling through eight code paths per tile (instruction-cache misses were the top stall,
// "no_instruction", in profiles/r01/ncu_table_scan_r01s4.txt).  The order inside a class is
// whatever the shared atomics give: each query's partials are still folded in tile and
// range order, so results do not depend on it.
__global__ void __launch_bounds__(1024) table_order_kernel(TableCols tc, int64_t nq, const TQuery* __restrict__ qs,
                                                           int32_t* __restrict__ perm) {
    __shared__ unsigned long long cnt[9];
    if (threadIdx.x < 9) cnt[threadIdx.x] = 0;
    __syncthreads();
    for (int64_t q = threadIdx.x; q < nq; q += blockDim.x) atomicAdd(&cnt[scan_class(tc, qs[q])], 1ull);
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long b = 0;
        for (int k = 0; k < 9; ++k) {
            const unsigned long long n = cnt[k];
            cnt[k] = b;
            b += n;
        }
    }
    __syncthreads();
    for (int64_t q = threadIdx.x; q < nq; q += blockDim.x)
        perm[atomicAdd(&cnt[scan_class(tc, qs[q])], 1ull)] = (int32_t)q;
}

// The shared scan, query-chunked.  The batch (in scan order) is cut into chunks of kChunkQ =
// 256 queries and the table into `nranges` contiguous tile ranges; block (range, chunk) -- the
// chunks of one range adjacent in blockIdx, so they run together and share each tile through
// L2 -- keeps its chunk's queries (SQ) and their partials in shared memory, stages its tiles
// one by one (every referenced column) and runs the chunk's queries on each, the warps claiming
// them one by one.  No per-(query, tile) global traffic; one partial per (range, query) at the
// end, folded in range order by table_final_kernel.
// OLAP_SCAN_MINBLOCKS: tuning knob (resident blocks per SM the register budget must allow).
constexpr int kChunkQ = kScanWarps * 32;
#ifdef OLAP_SCAN_MINBLOCKS
#define OLAP_SCAN_BOUNDS __launch_bounds__(kScanThreads, OLAP_SCAN_MINBLOCKS)
#else
#define OLAP_SCAN_BOUNDS __launch_bounds__(kScanThreads)
#endif
__global__ void OLAP_SCAN_BOUNDS table_scan_kernel(TableCols tc, int ncols, int64_t nrows, int64_t nq,
                                                   const TQuery* __restrict__ qs, TPartial* __restrict__ part,
                                                   const uint32_t* __restrict__ colmask,
                                                   const int32_t* __restrict__ perm, int nchunks,
                                                   int64_t tiles_per_range) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    SQ* sq = reinterpret_cast<SQ*>(smem_raw);                         // kChunkQ queries
    TPartial* acc = reinterpret_cast<TPartial*>(sq + kChunkQ);        // their partials
    int* ctr = reinterpret_cast<int*>(acc + kChunkQ);                 // per-tile claim counters (2)
    uint32_t* smem = reinterpret_cast<uint32_t*>(ctr + 4);            // ncols x kTileRows (the batch's columns)
    const uint32_t used = *colmask;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int chunk = (int)(blockIdx.x % (unsigned)nchunks);
    const int64_t range = blockIdx.x / (unsigned)nchunks;
    const int64_t ntiles = (nrows + kTileRows - 1) / kTileRows;
    const int64_t t0 = range * tiles_per_range, t1 = min(ntiles, t0 + tiles_per_range);
    // the chunk's queries in scan form
    for (int i = threadIdx.x; i < kChunkQ; i += kScanThreads) {
        const int64_t idx = (int64_t)chunk * kChunkQ + i;
        SQ d;
        memset(&d, 0, sizeof(d));
        d.ncond = -1;
        d.q = -1;
        if (idx < nq) {
            const int32_t q = perm[idx];
            const TQuery& t = qs[q];
            d.q = q;
            if (!t.flags && t.ncond >= 0) {
                d.ncond = t.ncond;
                const int opk = t.op == OLAP_MIN ? 1 : t.op == OLAP_MAX ? 2 : t.op == OLAP_COUNT ? 3 : 0;
                d.meta = t.data_col | (tc.dtype[t.data_col] == OLAP_FLOAT32 ? 1 : 0) << 8 | opk << 9;
                for (int k = 0; k < kInlineConds && k < t.ncond; ++k) {
                    d.colpack |= (uint32_t)t.c[k].col << (4 * k);
                    d.lo[k] = t.c[k].lo;
                    d.span[k] = t.c[k].span;
                }
            }
        }
        sq[i] = d;
    }
    // the chunk's partials live in shared memory; per tile, warps claim the chunk's queries one at
    // a time from a shared counter (ping-pong per tile parity), so uneven query costs balance
    // inside the tile and the barrier waits only for the last query
    for (int i = threadIdx.x; i < kChunkQ; i += kScanThreads) {
        acc[i].sum = 0;
        acc[i].count = 0;
        acc[i].code_max = INT_MIN;
        acc[i].code_min = INT_MIN;
    }
    if (threadIdx.x == 0) ctr[0] = ctr[1] = 0;
    const int nlive = (int)min((int64_t)kChunkQ, nq - (int64_t)chunk * kChunkQ);
    for (int64_t t = t0; t < t1; ++t) {
        const int64_t r0 = t * kTileRows;
        const int rows = (int)min((int64_t)kTileRows, nrows - r0);
        const int par = (int)(t & 1);
        __syncthreads();  // previous tile fully consumed (first pass: SQ, partials, counters written)
        for (int c = 0; c < ncols; ++c) {
            if (!((used >> c) & 1u)) continue;
            const uint32_t* src = tc.col[c] + r0;
            uint32_t* dst = smem + c * kTileRows;
            if (rows == kTileRows) {  // column starts are 256-B aligned: one 16-B load per thread
                static_assert(kTileRows == 4 * kScanThreads, "one uint4 per thread per column");
                reinterpret_cast<uint4*>(dst)[threadIdx.x] = __ldg(reinterpret_cast<const uint4*>(src) + threadIdx.x);
            } else {
                for (int r = threadIdx.x; r < rows; r += kScanThreads) dst[r] = __ldg(src + r);
            }
        }
        if (threadIdx.x == 0) ctr[par ^ 1] = 0;  // the next tile's counter (nobody claims from it now)
        __syncthreads();
        for (;;) {
            int i = 0;
            if (lane == 0) i = atomicAdd(&ctr[par], 1);
            i = __shfl_sync(0xffffffffu, i, 0);
            if (i >= nlive) break;
            const SQ* d = sq + i;
            const int32_t meta = d->meta;  // broadcast
            if (d->ncond < 0) continue;
            long long ts = 0;
            int32_t tn = 0, tmx = INT_MIN, tmn = INT_MIN;
            const int cls = meta >> 8;  // fl | opk << 1
            bool hit;
            switch (cls) {
                case 0: hit = scan_query_tile<false, 0>(smem, rows, d, qs, lane, ts, tn, tmx, tmn); break;
                case 2: hit = scan_query_tile<false, 1>(smem, rows, d, qs, lane, ts, tn, tmx, tmn); break;
                case 4: hit = scan_query_tile<false, 2>(smem, rows, d, qs, lane, ts, tn, tmx, tmn); break;
                case 6: hit = scan_query_tile<false, 3>(smem, rows, d, qs, lane, ts, tn, tmx, tmn); break;
                case 1: hit = scan_query_tile<true, 0>(smem, rows, d, qs, lane, ts, tn, tmx, tmn); break;
                case 3: hit = scan_query_tile<true, 1>(smem, rows, d, qs, lane, ts, tn, tmx, tmn); break;
                case 5: hit = scan_query_tile<true, 2>(smem, rows, d, qs, lane, ts, tn, tmx, tmn); break;
                default: hit = scan_query_tile<true, 3>(smem, rows, d, qs, lane, ts, tn, tmx, tmn); break;
            }
            if (hit && lane == 0) {  // one warp per (query, tile); tiles in order: deterministic
                TPartial& p = acc[i];
                p.sum = (cls & 1) ? __double_as_longlong(__longlong_as_double(p.sum) + __longlong_as_double(ts))
                                  : (long long)((unsigned long long)p.sum + (unsigned long long)ts);
                p.count += tn;
                p.code_max = max(p.code_max, tmx);
                p.code_min = max(p.code_min, tmn);
            }
        }
    }
    __syncthreads();
    for (int i = threadIdx.x; i < nlive; i += kScanThreads)
        if (sq[i].q >= 0) part[range * nq + sq[i].q] = acc[i];
}

// fold per-range partials in range order -> results
__global__ void table_final_kernel(TableCols tc, int64_t nq, int nblocks, const TQuery* __restrict__ qs,
                                   const TPartial* __restrict__ part, olap_result* __restrict__ out) {
    const int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (q >= nq) return;
    const TQuery& tq = qs[q];
    olap_result r;
    r.i = 0;
    r.d = 0.0;
    r.flags = 0;
    r._pad = 0;
    if (tq.flags) {
        r.flags = OLAP_RESULT_INVALID;
        out[q] = r;
        return;
    }
    const bool fl = tc.dtype[tq.data_col] == OLAP_FLOAT32;
    long long s = 0;
    int64_t cnt = 0;
    int32_t cmx = INT_MIN, cmn = INT_MIN;
    if (tq.ncond >= 0) {
        for (int b = 0; b < nblocks; ++b) {
            const TPartial p = part[(int64_t)b * nq + q];
            s = fl ? __double_as_longlong(__longlong_as_double(s) + __longlong_as_double(p.sum))
                   : (long long)((unsigned long long)s + (unsigned long long)p.sum);
            cnt += p.count;
            cmx = max(cmx, p.code_max);
            cmn = max(cmn, p.code_min);
        }
    }
    if (cnt == 0) {
        r.flags = OLAP_RESULT_EMPTY;
    } else if (tq.op == OLAP_COUNT) {
        r.i = cnt;
    } else if (!fl) {
        if (tq.op == OLAP_SUM) r.i = s;
        else if (tq.op == OLAP_MIN) r.i = ~cmn;
        else if (tq.op == OLAP_MAX) r.i = cmx;
        else r.d = (double)s / (double)cnt;
    } else {
        const double ds = __longlong_as_double(s);
        if (tq.op == OLAP_SUM) r.d = ds;
        else if (tq.op == OLAP_MIN) r.d = (double)tf32_decode(~cmn);
        else if (tq.op == OLAP_MAX) r.d = (double)tf32_decode(cmx);
        else r.d = ds / (double)cnt;
    }
    out[q] = r;
}

}  // namespace olap

using namespace olap;

// Launch workspace: per-query descriptors and per-(block, query) partials.  The table's
// own calls use one; every partition (olap_table_part) has its own, so partitions run
// concurrently.
struct TWork {
    int sm_count = 0, blocks = 0;
    int64_t nq_cap = 0;
    TQuery* d_qs = nullptr;
    TPartial* d_part = nullptr;
    uint32_t* d_colmask = nullptr;
    int32_t* d_perm = nullptr;  // batch order grouped by scan instantiation (table_order_kernel)
    cudaEvent_t done = nullptr; // recorded after the last kernel of every batch on this workspace: a
                                // batch on another stream waits for it before touching d_qs / d_part
    std::mutex mu;
};

struct olap_table {
    int device = 0;
    int64_t nrows = 0;
    int ncols = 0;
    int32_t dtype[kMaxTableCols] = {};
    void* d_data = nullptr;      // all columns one after another, 256-B aligned
    int64_t col_stride = 0;      // cells between column starts
    std::mutex mu;               // host staging buffers below
    cudaStream_t stream = nullptr;
    int num_sms = 0, blocks_per_sm = 0;
    TWork work;
    olap_result* d_res = nullptr;
    int64_t res_cap = 0;
    olap_cond* d_conds = nullptr;
    int64_t conds_cap = 0;
    int64_t* d_off = nullptr;
    int32_t* d_dcol = nullptr;
    int32_t* d_ops = nullptr;
    int64_t launches = 0;
    // olap_table_profile: CUDA events around every table_scan_kernel launch of the table's own calls
    bool prof = false;
    std::vector<cudaEvent_t> ev;
    size_t ev_used = 0;
};

struct olap_table_part {
    olap_table* t = nullptr;
    TWork work;
};

namespace {

size_t scan_smem_bytes(int ncols) {
    return (sizeof(SQ) + sizeof(TPartial)) * kChunkQ + 4 * sizeof(int) + sizeof(uint32_t) * kTileRows * ncols;
}

struct TDevGuard {
    int prev = -1;
    explicit TDevGuard(int dev) {
        if (cudaGetDevice(&prev) == cudaSuccess) cudaSetDevice(dev);
    }
    ~TDevGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

TableCols cols_of(const olap_table* t) {
    TableCols tc;
    std::memset(&tc, 0, sizeof(tc));
    for (int c = 0; c < t->ncols; ++c) {
        tc.col[c] = static_cast<const uint32_t*>(t->d_data) + c * t->col_stride;
        tc.dtype[c] = t->dtype[c];
    }
    return tc;
}

void free_work(TWork& w) {
    cudaFree(w.d_qs);
    cudaFree(w.d_part);
    cudaFree(w.d_colmask);
    cudaFree(w.d_perm);
    w.d_perm = nullptr;
    w.d_qs = nullptr;
    w.d_part = nullptr;
    w.d_colmask = nullptr;
    w.nq_cap = 0;
    if (w.done) cudaEventDestroy(w.done);
    w.done = nullptr;
}

void init_work(const olap_table* t, TWork& w, int sm_count) {
    w.sm_count = (sm_count <= 0 || sm_count > t->num_sms) ? t->num_sms : sm_count;
    w.blocks = w.sm_count * std::max(t->blocks_per_sm, 1);
}

bool stream_capturing(cudaStream_t st) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    return cudaStreamIsCapturing(st, &cs) == cudaSuccess && cs == cudaStreamCaptureStatusActive;
}

// (re)size a workspace and order `st` after the workspace's previous batch, whatever stream
// that batch ran on (w.done); the caller records w.done on `st` after its last kernel
int ensure_work(TWork& w, int64_t nq, cudaStream_t st) {
    if (!w.d_colmask) OLAP_CUDA_TRY(cudaMalloc(&w.d_colmask, sizeof(uint32_t)));
    if (!w.done) OLAP_CUDA_TRY(cudaEventCreateWithFlags(&w.done, cudaEventDisableTiming));
    if (nq > w.nq_cap) {
        if (stream_capturing(st))
            return set_error(OLAP_E_STATE, "stream capture: run one batch of %lld queries outside capture first",
                             (long long)nq);
        OLAP_CUDA_TRY(cudaEventSynchronize(w.done));
        cudaFree(w.d_qs);
        cudaFree(w.d_part);
        cudaFree(w.d_perm);
        w.d_qs = nullptr;
        w.d_part = nullptr;
        w.d_perm = nullptr;
        w.nq_cap = 0;
        const int64_t cap = std::max<int64_t>(nq, 256);
        OLAP_CUDA_TRY(cudaMalloc(&w.d_qs, sizeof(TQuery) * cap));
        OLAP_CUDA_TRY(cudaMalloc(&w.d_part, sizeof(TPartial) * cap * w.blocks));
        OLAP_CUDA_TRY(cudaMalloc(&w.d_perm, sizeof(int32_t) * cap));
        w.nq_cap = cap;
    }
    if (!stream_capturing(st)) OLAP_CUDA_TRY(cudaStreamWaitEvent(st, w.done, 0));
    return OLAP_OK;
}

int ensure_staging(olap_table* t, int64_t nq, int64_t nconds) {
    if (nq > t->res_cap) {
        OLAP_CUDA_TRY(cudaStreamSynchronize(t->stream));
        cudaFree(t->d_off);
        cudaFree(t->d_dcol);
        cudaFree(t->d_ops);
        cudaFree(t->d_res);
        t->d_off = nullptr;
        t->d_dcol = nullptr;
        t->d_ops = nullptr;
        t->d_res = nullptr;
        t->res_cap = 0;
        const int64_t cap = std::max<int64_t>(nq, 256);
        OLAP_CUDA_TRY(cudaMalloc(&t->d_off, sizeof(int64_t) * (cap + 1)));
        OLAP_CUDA_TRY(cudaMalloc(&t->d_dcol, sizeof(int32_t) * cap));
        OLAP_CUDA_TRY(cudaMalloc(&t->d_ops, sizeof(int32_t) * cap));
        OLAP_CUDA_TRY(cudaMalloc(&t->d_res, sizeof(olap_result) * cap));
        t->res_cap = cap;
    }
    if (nconds > t->conds_cap) {
        OLAP_CUDA_TRY(cudaStreamSynchronize(t->stream));
        cudaFree(t->d_conds);
        t->d_conds = nullptr;
        t->conds_cap = 0;
        const int64_t cap = std::max<int64_t>(nconds, 1024);
        OLAP_CUDA_TRY(cudaMalloc(&t->d_conds, sizeof(olap_cond) * cap));
        t->conds_cap = cap;
    }
    return OLAP_OK;
}

// scan + fold, after a prep kernel has written w.d_qs and w.d_colmask on `st`
int launch_scan_fold(olap_table* t, TWork& w, int64_t nq, olap_result* d_res, cudaStream_t st) {
    const TableCols tc = cols_of(t);
    const size_t smem = scan_smem_bytes(t->ncols);
    if (nq > INT32_MAX) return set_error(OLAP_E_INVALID, "table batch of %lld queries: at most 2^31-1", (long long)nq);
    // (range, chunk) blocks: one resident wave when the batch has at most w.blocks chunks
    const int64_t nchunks = (nq + kChunkQ - 1) / kChunkQ;
    if (nchunks > INT32_MAX / 2) return set_error(OLAP_E_INVALID, "table batch too large");
    const int64_t ntiles = (t->nrows + kTileRows - 1) / kTileRows;
    int64_t nranges = std::max<int64_t>(1, w.blocks / nchunks);
    nranges = std::min(nranges, ntiles);
    const int64_t per = (ntiles + nranges - 1) / nranges;
    nranges = (ntiles + per - 1) / per;
    const int64_t grid = nranges * nchunks;
    if (grid > INT32_MAX) return set_error(OLAP_E_INVALID, "table batch too large");
    table_order_kernel<<<1, 1024, 0, st>>>(tc, nq, w.d_qs, w.d_perm);
    const bool prof = t->prof && &w == &t->work && !stream_capturing(st);
    if (prof) {
        while (t->ev.size() < t->ev_used + 2) {
            cudaEvent_t e;
            OLAP_CUDA_TRY(cudaEventCreate(&e));
            t->ev.push_back(e);
        }
        OLAP_CUDA_TRY(cudaEventRecord(t->ev[t->ev_used], st));
    }
    table_scan_kernel<<<(unsigned)grid, kScanThreads, smem, st>>>(tc, t->ncols, t->nrows, nq, w.d_qs, w.d_part,
                                                                   w.d_colmask, w.d_perm, (int)nchunks, per);
    if (prof) {
        OLAP_CUDA_TRY(cudaEventRecord(t->ev[t->ev_used + 1], st));
        t->ev_used += 2;
    }
    table_final_kernel<<<(int)((nq + 255) / 256), 256, 0, st>>>(tc, nq, (int)nranges, w.d_qs, w.d_part, d_res);
    OLAP_CUDA_TRY(cudaGetLastError());
    if (!stream_capturing(st)) OLAP_CUDA_TRY(cudaEventRecord(w.done, st));
    __atomic_fetch_add(&t->launches, 4, __ATOMIC_RELAXED);
    return OLAP_OK;
}

int launch_scan(olap_table* t, TWork& w, int64_t nq, const int64_t* d_off, const olap_cond* d_conds,
                const int32_t* d_dcol, const int32_t* d_ops, olap_result* d_res, cudaStream_t st) {
    const TableCols tc = cols_of(t);
    OLAP_CUDA_TRY(cudaMemsetAsync(w.d_colmask, 0, sizeof(uint32_t), st));
    table_prep_kernel<<<(int)((nq + 255) / 256), 256, 0, st>>>(nq, t->ncols, tc, d_off, d_conds, d_dcol, d_ops,
                                                               w.d_qs, w.d_colmask);
    return launch_scan_fold(t, w, nq, d_res, st);
}

int launch_scan_boxes(olap_table* t, TWork& w, int64_t nq, const BoxMap& bm, const olap_range* d_boxes,
                      const int32_t* d_dcol, const int32_t* d_ops, olap_result* d_res, cudaStream_t st) {
    const TableCols tc = cols_of(t);
    OLAP_CUDA_TRY(cudaMemsetAsync(w.d_colmask, 0, sizeof(uint32_t), st));
    table_prep_boxes_kernel<<<(int)((nq + 255) / 256), 256, 0, st>>>(nq, t->ncols, tc, bm, d_boxes, d_dcol, d_ops,
                                                                     w.d_qs, w.d_colmask);
    return launch_scan_fold(t, w, nq, d_res, st);
}

}  // namespace

extern "C" {

int olap_table_create(int64_t nrows, int ncols, const int32_t* dtypes, int device, olap_table** out) {
    clear_error();
    if (!out || !dtypes) return set_error(OLAP_E_INVALID, "olap_table_create: NULL argument");
    if (nrows < 1) return set_error(OLAP_E_INVALID, "nrows < 1");
    if (ncols < 1 || ncols > kMaxTableCols) return set_error(OLAP_E_INVALID, "ncols %d not in [1,16]", ncols);
    for (int c = 0; c < ncols; ++c)
        if (dtypes[c] != OLAP_INT32 && dtypes[c] != OLAP_FLOAT32)
            return set_error(OLAP_E_INVALID, "column %d: bad dtype %d", c, dtypes[c]);
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
        return set_error(OLAP_E_CUDA, "no CUDA device available (the library has no CPU fallback)");
    if (device < 0 || device >= ndev) return set_error(OLAP_E_INVALID, "device %d not in [0,%d)", device, ndev);
    TDevGuard g(device);
    olap_table* t = new (std::nothrow) olap_table();
    if (!t) return set_error(OLAP_E_NOMEM, "host allocation failed");
    t->device = device;
    t->nrows = nrows;
    t->ncols = ncols;
    for (int c = 0; c < ncols; ++c) t->dtype[c] = dtypes[c];
    t->col_stride = (nrows + 63) & ~63ll;  // 256-B aligned column starts
    cudaError_t e = cudaMalloc(&t->d_data, sizeof(uint32_t) * t->col_stride * ncols);
    if (e != cudaSuccess) {
        cudaGetLastError();
        delete t;
        return set_error(e == cudaErrorMemoryAllocation ? OLAP_E_NOMEM : OLAP_E_CUDA, "table allocation: %s",
                         cudaGetErrorString(e));
    }
    cudaStreamCreateWithFlags(&t->stream, cudaStreamNonBlocking);
    cudaDeviceGetAttribute(&t->num_sms, cudaDevAttrMultiProcessorCount, device);
    const size_t smem = scan_smem_bytes(ncols);
    if (smem > 48 * 1024)
        cudaFuncSetAttribute(table_scan_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int bps = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, table_scan_kernel, kScanThreads, smem);
    t->blocks_per_sm = std::max(bps, 1);
    init_work(t, t->work, 0);
    *out = t;
    return OLAP_OK;
}

int olap_table_load_column(olap_table* t, int col, const void* values) {
    clear_error();
    if (!t || !values) return set_error(OLAP_E_INVALID, "NULL argument");
    if (col < 0 || col >= t->ncols) return set_error(OLAP_E_INVALID, "column %d not in [0,%d)", col, t->ncols);
    std::lock_guard<std::mutex> lk(t->mu);
    TDevGuard g(t->device);
    OLAP_CUDA_TRY(cudaMemcpy(static_cast<uint32_t*>(t->d_data) + col * t->col_stride, values,
                             sizeof(uint32_t) * t->nrows, cudaMemcpyHostToDevice));
    return OLAP_OK;
}

int olap_table_column_device(olap_table* t, int col, void** d_ptr) {
    clear_error();
    if (!t || !d_ptr) return set_error(OLAP_E_INVALID, "NULL argument");
    if (col < 0 || col >= t->ncols) return set_error(OLAP_E_INVALID, "column %d not in [0,%d)", col, t->ncols);
    *d_ptr = static_cast<uint32_t*>(t->d_data) + col * t->col_stride;
    return OLAP_OK;
}

int olap_table_query_batch_device(olap_table* t, int64_t nq, const int64_t* d_cond_offsets, const olap_cond* d_conds,
                                  const int32_t* d_data_cols, const int32_t* d_ops, olap_result* d_results,
                                  void* stream) {
    clear_error();
    if (!t) return set_error(OLAP_E_INVALID, "table handle is NULL");
    if (nq < 0) return set_error(OLAP_E_INVALID, "nq < 0");
    if (nq == 0) return OLAP_OK;
    if (!d_cond_offsets || !d_data_cols || !d_ops || !d_results) return set_error(OLAP_E_INVALID, "NULL device buffer");
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    std::lock_guard<std::mutex> lk(t->work.mu);
    TDevGuard g(t->device);
    int rc = ensure_work(t->work, nq, st);
    if (rc) return rc;
    return launch_scan(t, t->work, nq, d_cond_offsets, d_conds, d_data_cols, d_ops, d_results, st);
}

int olap_table_query_batch(olap_table* t, int64_t nq, const int64_t* cond_offsets, const olap_cond* conds,
                           const int32_t* data_cols, const int32_t* ops, olap_result* results) {
    clear_error();
    if (!t) return set_error(OLAP_E_INVALID, "table handle is NULL");
    if (nq < 0) return set_error(OLAP_E_INVALID, "nq < 0");
    if (nq == 0) return OLAP_OK;
    if (!cond_offsets || !data_cols || !ops || !results) return set_error(OLAP_E_INVALID, "NULL buffer");
    if (cond_offsets[0] != 0) return set_error(OLAP_E_INVALID, "cond_offsets[0] must be 0");
    for (int64_t q = 0; q < nq; ++q) {
        const int64_t n = cond_offsets[q + 1] - cond_offsets[q];
        if (n < 0 || n > kMaxConds)
            return set_error(OLAP_E_INVALID, "query %lld: %lld conditions (max 16)", (long long)q, (long long)n);
        if (ops[q] < OLAP_SUM || ops[q] > OLAP_AVG)
            return set_error(OLAP_E_INVALID, "query %lld: unknown op %d", (long long)q, ops[q]);
        if (data_cols[q] < 0 || data_cols[q] >= t->ncols)
            return set_error(OLAP_E_INVALID, "query %lld: data column %d", (long long)q, data_cols[q]);
        for (int64_t k = cond_offsets[q]; k < cond_offsets[q + 1]; ++k)
            if (conds[k].col < 0 || conds[k].col >= t->ncols || t->dtype[conds[k].col] != OLAP_INT32)
                return set_error(OLAP_E_INVALID, "query %lld: condition on column %d (must be an int32 column)",
                                 (long long)q, conds[k].col);
    }
    const int64_t nconds = cond_offsets[nq];
    std::lock_guard<std::mutex> lk(t->mu);
    std::lock_guard<std::mutex> lw(t->work.mu);
    TDevGuard g(t->device);
    cudaStream_t st = t->stream;
    int rc = ensure_staging(t, nq, nconds);
    if (rc) return rc;
    rc = ensure_work(t->work, nq, st);
    if (rc) return rc;
    OLAP_CUDA_TRY(cudaMemcpyAsync(t->d_off, cond_offsets, sizeof(int64_t) * (nq + 1), cudaMemcpyHostToDevice, st));
    if (nconds)
        OLAP_CUDA_TRY(cudaMemcpyAsync(t->d_conds, conds, sizeof(olap_cond) * nconds, cudaMemcpyHostToDevice, st));
    OLAP_CUDA_TRY(cudaMemcpyAsync(t->d_dcol, data_cols, sizeof(int32_t) * nq, cudaMemcpyHostToDevice, st));
    OLAP_CUDA_TRY(cudaMemcpyAsync(t->d_ops, ops, sizeof(int32_t) * nq, cudaMemcpyHostToDevice, st));
    rc = launch_scan(t, t->work, nq, t->d_off, t->d_conds, t->d_dcol, t->d_ops, t->d_res, st);
    if (rc) return rc;
    OLAP_CUDA_TRY(cudaMemcpyAsync(results, t->d_res, sizeof(olap_result) * nq, cudaMemcpyDeviceToHost, st));
    OLAP_CUDA_TRY(cudaStreamSynchronize(st));
    return OLAP_OK;
}

int olap_table_profile(olap_table* t, int enable) {
    clear_error();
    if (!t) return set_error(OLAP_E_INVALID, "table handle is NULL");
    std::lock_guard<std::mutex> lk(t->work.mu);
    TDevGuard g(t->device);
    if (t->work.done) OLAP_CUDA_TRY(cudaEventSynchronize(t->work.done));
    t->prof = enable != 0;
    t->ev_used = 0;
    return OLAP_OK;
}

int olap_table_profile_read(olap_table* t, double* scan_ms, int64_t* launches) {
    clear_error();
    if (!t) return set_error(OLAP_E_INVALID, "table handle is NULL");
    std::lock_guard<std::mutex> lk(t->work.mu);
    TDevGuard g(t->device);
    double ms = 0.0;
    for (size_t i = 0; i + 1 < t->ev_used; i += 2) {
        float x = 0.f;
        OLAP_CUDA_TRY(cudaEventSynchronize(t->ev[i + 1]));
        OLAP_CUDA_TRY(cudaEventElapsedTime(&x, t->ev[i], t->ev[i + 1]));
        ms += x;
    }
    if (scan_ms) *scan_ms = ms;
    if (launches) *launches = (int64_t)(t->ev_used / 2);
    return OLAP_OK;
}

int olap_table_destroy(olap_table* t) {
    clear_error();
    if (!t) return OLAP_OK;
    TDevGuard g(t->device);
    cudaDeviceSynchronize();  // the table's and its partitions' launches (any stream)
    for (auto e : t->ev) cudaEventDestroy(e);
    free_work(t->work);
    cudaFree(t->d_off);
    cudaFree(t->d_dcol);
    cudaFree(t->d_ops);
    cudaFree(t->d_res);
    cudaFree(t->d_conds);
    cudaFree(t->d_data);
    if (t->stream) cudaStreamDestroy(t->stream);
    delete t;
    return OLAP_OK;
}

int olap_table_part_create(olap_table* t, int sm_count, olap_table_part** out) {
    clear_error();
    if (!t || !out) return set_error(OLAP_E_INVALID, "NULL argument");
    olap_table_part* p = new (std::nothrow) olap_table_part();
    if (!p) return set_error(OLAP_E_NOMEM, "host allocation failed");
    p->t = t;
    init_work(t, p->work, sm_count);
    *out = p;
    return OLAP_OK;
}

int olap_table_part_sms(const olap_table_part* p, int* sm_count, int* blocks) {
    clear_error();
    if (!p) return set_error(OLAP_E_INVALID, "NULL argument");
    if (sm_count) *sm_count = p->work.sm_count;
    if (blocks) *blocks = p->work.blocks;
    return OLAP_OK;
}

int olap_table_part_query_device(olap_table_part* p, int64_t nq, const int64_t* d_cond_offsets,
                                 const olap_cond* d_conds, const int32_t* d_data_cols, const int32_t* d_ops,
                                 olap_result* d_results, void* stream) {
    clear_error();
    if (!p) return set_error(OLAP_E_INVALID, "partition handle is NULL");
    if (nq < 0) return set_error(OLAP_E_INVALID, "nq < 0");
    if (nq == 0) return OLAP_OK;
    if (!d_cond_offsets || !d_data_cols || !d_ops || !d_results) return set_error(OLAP_E_INVALID, "NULL device buffer");
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    std::lock_guard<std::mutex> lk(p->work.mu);
    TDevGuard g(p->t->device);
    int rc = ensure_work(p->work, nq, st);
    if (rc) return rc;
    return launch_scan(p->t, p->work, nq, d_cond_offsets, d_conds, d_data_cols, d_ops, d_results, st);
}

int olap_table_part_query_boxes_device(olap_table_part* p, int64_t nq, int ndims, const int32_t* dim_cols,
                                       const int64_t* extents, const olap_range* d_boxes,
                                       const int32_t* d_data_cols, const int32_t* d_ops, olap_result* d_results,
                                       void* stream) {
    clear_error();
    if (!p) return set_error(OLAP_E_INVALID, "partition handle is NULL");
    if (nq < 0) return set_error(OLAP_E_INVALID, "nq < 0");
    if (nq == 0) return OLAP_OK;
    if (ndims < 1 || ndims > kMaxConds) return set_error(OLAP_E_INVALID, "ndims %d not in [1,16]", ndims);
    if (!dim_cols || !extents || !d_boxes || !d_data_cols || !d_ops || !d_results)
        return set_error(OLAP_E_INVALID, "NULL buffer");
    olap_table* t = p->t;
    BoxMap bm;
    std::memset(&bm, 0, sizeof(bm));
    bm.ndims = ndims;
    for (int d = 0; d < ndims; ++d) {
        if (dim_cols[d] < 0 || dim_cols[d] >= t->ncols || t->dtype[dim_cols[d]] != OLAP_INT32)
            return set_error(OLAP_E_INVALID, "dimension %d: column %d is not an int32 column", d, dim_cols[d]);
        if (extents[d] < 1) return set_error(OLAP_E_INVALID, "dimension %d: extent < 1", d);
        bm.col[d] = dim_cols[d];
        bm.extent[d] = extents[d];
    }
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    std::lock_guard<std::mutex> lk(p->work.mu);
    TDevGuard g(t->device);
    int rc = ensure_work(p->work, nq, st);
    if (rc) return rc;
    return launch_scan_boxes(t, p->work, nq, bm, d_boxes, d_data_cols, d_ops, d_results, st);
}

int olap_table_part_destroy(olap_table_part* p) {
    clear_error();
    if (!p) return OLAP_OK;
    TDevGuard g(p->t->device);
    cudaDeviceSynchronize();
    free_work(p->work);
    delete p;
    return OLAP_OK;
}

}  // extern "C"
