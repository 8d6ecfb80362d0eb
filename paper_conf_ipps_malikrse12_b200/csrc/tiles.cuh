// tiles.cuh — the tile-shared scan (included by cube.cu; internal, not part of the C-ABI).
//
// The item path (reduce_kernel) streams every query's own bytes through L1TEX from L2.
// When a batch's boxes overlap heavily (C2a: every cell is read by ~390 queries of a
// 4,096-query batch), that costs the same on-chip bandwidth 390 times over.  This path
// reorganises the same reduction (Fig. 2 "area of limited search", PAPER.md:143,151;
// bandwidth-bound) around the cube instead of around the queries:
//
//   * the cube is cut into TILES: contiguous spans that are also boxes,
//     (1, .., 1, ct, n_{kt+1}, .., n_{N-1}) cells, <= 64 KiB;
//   * a (query, tile) PAIR is a query box intersecting a tile; its cells are the box
//     clipped to the tile, again runs of the row-major layout (a4);
//   * a persistent block per SM pops non-empty tiles, stages each one into shared memory
//     ONCE with a bulk async copy (cp.async.bulk + mbarrier, 3-stage ring fed by a
//     producer warp), and its 31 consumer warps reduce every pair of that tile from shared
//     memory, each pair with the item path's run streamer (LDS instead of LDG);
//   * pair partials are stored by pair id (query-major) and folded per query in pair
//     order, so results are deterministic and independent of the tile schedule.
//
// Planning (all on the device, capturable): tile_desc_kernel (per query: tile box, pair
// count, clipped-run structure) -> tile_scan_kernel (pair offsets; chooses this path or
// the item path from the batch's reuse) -> tile_count_kernel ->
// exclusive scan of per-tile counts (CUB) -> tile_scatter_kernel (per-tile query lists)
// -> tile_reduce_kernel -> pair_fold_kernel.  Every kernel of the path not chosen exits
// at once.

#ifndef OLAP_TILE_CELLS_F
#define OLAP_TILE_CELLS_F 16384
#endif
#ifndef OLAP_TILE_CELLS_I
#define OLAP_TILE_CELLS_I 12288
#endif
#ifndef OLAP_TILE_NO_SUMMARY
#define OLAP_TILE_NO_SUMMARY 0  // 1: every pair through the item-path streamers (A/B of the summary path)
#endif
#ifndef OLAP_TILE_STAGES
#define OLAP_TILE_STAGES 2
#endif
// Cells per tile: 64 KiB for float32 cubes, 48 KiB for int32 (whose SUM trees hold int64 entries):
// two stages of cells + slot trees fill the 227 KiB of shared memory.  Fewer, bigger tiles mean fewer
// (query, tile) pairs, and the per-pair set-up is a large part of the work (32-KiB tiles: C2a -22%).
constexpr int64_t kTileCellsF = OLAP_TILE_CELLS_F, kTileCellsI = OLAP_TILE_CELLS_I;
__host__ __device__ constexpr int64_t tile_cells_max(bool is_float) { return is_float ? kTileCellsF : kTileCellsI; }
constexpr int kTileStages = OLAP_TILE_STAGES;
#ifndef OLAP_TILE_WARPS
#define OLAP_TILE_WARPS 32
#endif
constexpr int kTileWarps = OLAP_TILE_WARPS;  // warp 0: producer; warps 1..: consumers
constexpr int kTileThreads = kTileWarps * 32;
constexpr int kTileConsumers = kTileWarps - 1;
constexpr int kTileSlack = 16;  // cells after each stage buffer: masked over-reads of a run's last slot
constexpr int kTilePairsPerThread = 8;
constexpr int kTreeTop = 5;  // slot trees (below): highest level, blocks of 32 slots (256 cells)

// Tile geometry of a cube (shard-local), fixed at cube creation.
struct TGeo {
    int nd, kt, padded, ok;
    int64_t ct, nct, ntiles, tcells;  // chunk extent along kt, chunks, tiles, cells of a full tile
    int64_t ext[kMaxDims];            // local extents (dim 0 = local rows)
    int64_t stride[kMaxDims];         // local strides (cells)
    int64_t ts[kMaxDims];             // tile-grid strides for dims <= kt
};

// Per query: its tile box and the part of its clipped-run structure that no tile changes.
struct TDesc {
    int32_t opc, V, nrd, span;  // span: a pair is one run over dim kt (all dims after kt full)
    int64_t lo_kt, hi_kt;       // local range along kt
    int64_t L, Rin, base_in;    // run length, runs per kt-slice, offset of dims > kt
    int64_t tlo[kMaxDims];      // tile box: dims < kt: lo_e; dim kt: first chunk
    int64_t tn[kMaxDims];       // tile box extents
    FastDiv tfd[kMaxDims];      // / tn (pair index -> tile coordinates)
    FastDiv frl[kMaxRunDims];   // inner radices (dims ks-1 .. kt+1 with extent > 1), innermost first
    int64_t rs[kMaxRunDims];
};

// Per query, the compact descriptor of the summary path (one 128-B line: 32 words, loaded by the
// 32 lanes of a warp in one coalesced request and broadcast with shuffles).  Valid (mode = 1) when
// every run starts 32-B aligned modulo one shared offset h0 (V = 8) and a pair's runs need at most
// one digit besides dim kt's.  Inside a tile everything fits 32-bit arithmetic.
struct SDesc {
    int32_t mode, opc, span, Lin;   // Lin: run length (cells) when not span
    int32_t rad, rs, skt, lo_kt;    // inner digit radix (1: none) and stride; stride of dim kt; local range
    int32_t hi_kt, base_in, jbase, radm;  // offset of dims > kt; pair index base; fast-div magic of rad
    int32_t radl, nkt, npat, pad1;        // fast-div shift; dims < kt used in tstr; pattern length (-1: none)
    int32_t tstr[8];                      // tile-box strides of dims < kt (pair index j)
    uint16_t pat[16];                     // the run interior's tree entries: level << 13 | node offset
};
static_assert(sizeof(SDesc) == 128, "one line per query");

// A run of L cells starting at cell h0 of its first 8-cell slot covers nslot slots.  Its tree
// interior is slots [i0, i1) -- every FULL slot, the first and last included when they are
// whole -- and its edge cells are E1 cells of a partial first slot (h0 ..) and E2 of a partial
// last slot (0 .. E2-1).
struct RunSplit {
    uint32_t nslot, i0, i1, E1, E2;
};
__host__ __device__ __forceinline__ RunSplit run_split(uint32_t h0, uint32_t L) {
    RunSplit r;
    r.nslot = (h0 + L + 7) >> 3;
    if (r.nslot == 1) {
        const bool full = L == 8;  // h0 = 0
        r.i0 = full ? 0u : 1u;
        r.i1 = full ? 1u : 0u;
        r.E1 = full ? 0u : L;
        r.E2 = 0;
    } else {
        const uint32_t tail = h0 + L - 8 * (r.nslot - 1);
        r.i0 = h0 ? 1u : 0u;
        r.i1 = r.nslot - (tail < 8 ? 1u : 0u);
        r.E1 = h0 ? 8 - h0 : 0u;
        r.E2 = tail < 8 ? tail : 0u;
    }
    return r;
}


// ------------------------------------------------------------------ mbarrier / bulk copy (PTX)

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
// A wait that never completes is a bug (a phase nobody will reach); rather than hang the GPU, a
// waiter that has waited ~8 s traps the kernel (cudaErrorLaunchFailure: an error, not a hang).
constexpr long long kWaitTrapCycles = 16ll * 1000 * 1000 * 1000;
__device__ __forceinline__ bool mbar_try(uint64_t* b, uint32_t parity) {
    uint32_t ok = 0;
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
        "selp.u32 %0, 1, 0, p;\n"
        "}\n"
        : "=r"(ok)
        : "r"(smem_u32(b)), "r"(parity)
        : "memory");
    return ok != 0;
}
// try_wait with a suspend-time hint: the warp is suspended in hardware until the phase completes
// (or the hint expires) instead of spinning on the issue slots the reducing warps need (a spin
// loop with __nanosleep took 13% of the kernel's instructions once the consumers got faster)
__device__ __forceinline__ bool mbar_try_suspend(uint64_t* b, uint32_t parity, uint32_t hint_ns) {
    uint32_t ok = 0;
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n"
        "selp.u32 %0, 1, 0, p;\n"
        "}\n"
        : "=r"(ok)
        : "r"(smem_u32(b)), "r"(parity), "r"(hint_ns)
        : "memory");
    return ok != 0;
}
#ifndef OLAP_WAIT_HINT_NS
#define OLAP_WAIT_HINT_NS 1000000u
#endif
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
    if (mbar_try(b, parity)) return;  // the common case: one probe
    const long long t0 = clock64();
    for (;;) {
        if (mbar_try_suspend(b, parity, OLAP_WAIT_HINT_NS)) return;
        if (clock64() - t0 > kWaitTrapCycles) __trap();
    }
}
// producer side: the same wait
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* b, uint32_t parity) { mbar_wait(b, parity); }
// global -> shared bulk copy completing on mbarrier b (bytes: multiple of 16, both ends 16-B aligned)
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(b))
                 : "memory");
}

// ------------------------------------------------------------------ planning

// One thread per query: validate (a1), shard-intersect (a3), tile box, pair count, clipped-run
// structure; identity partials for queries that read no cell; batch totals (order-free atomics).
__global__ void __launch_bounds__(kDescThreads) tile_desc_kernel(Geo geo, TGeo tg, int64_t nq,
                                                                 const olap_range* __restrict__ ranges,
                                                                 const int32_t* __restrict__ ops, TDesc* tdesc,
                                                                 SDesc* sdesc, int64_t* q_pairs, int64_t* psum,
                                                                 int32_t* pext, unsigned long long* totals) {
    __shared__ int64_t sh[32];
    const int64_t q = blockIdx.x * (int64_t)kDescThreads + threadIdx.x;
    int64_t cells = 0;
    if (q < nq) {
        int64_t np = 0;
        const int32_t op = ops[q];
        int64_t lo[kMaxDims], hi[kMaxDims];
        bool ok = op >= OLAP_SUM && op <= OLAP_AVG && op != OLAP_COUNT, empty = false;
        for (int k = 0; k < geo.nd && ok; ++k) {
            lo[k] = ranges[q * geo.nd + k].lo;
            hi[k] = ranges[q * geo.nd + k].hi;
            if (lo[k] < 0 || hi[k] >= geo.n[k]) ok = false;
            if (lo[k] > hi[k]) empty = true;
        }
        if (ok && !empty) {
            int64_t llo, lhi;
            if (shard_local_range(geo.n[0], geo.G, geo.g, geo.b, lo[0], hi[0], &llo, &lhi)) {
                lo[0] = llo;
                hi[0] = lhi;
            } else {
                ok = false;
            }
        }
        if (ok && !empty) {
            TDesc d;
            const int nd = tg.nd, kt = tg.kt;
            int64_t ell[kMaxDims];
            cells = 1;
            for (int k = 0; k < nd; ++k) {
                ell[k] = hi[k] - lo[k] + 1;
                cells *= ell[k];
            }
            d.opc = (op == OLAP_MIN) ? OPC_MIN : (op == OLAP_MAX) ? OPC_MAX : OPC_SUM;
            d.lo_kt = lo[kt];
            d.hi_kt = hi[kt];
            // split dim among dims > kt: innermost not fully covered (never merge across padded rows)
            int ks = nd - 1;
            if (kt == nd - 1) {
                ks = kt;
            } else if (!tg.padded) {
                while (ks > kt && ell[ks] == tg.ext[ks]) --ks;
            }
            d.span = ks == kt;
            d.base_in = 0;
            for (int k = kt + 1; k < nd; ++k) d.base_in += lo[k] * tg.stride[k];
            bool a8 = (tg.stride[kt] & 7) == 0 || d.span, a4 = (tg.stride[kt] & 3) == 0 || d.span;
            int nrd = 0;
            d.Rin = 1;
            d.L = 0;
            if (!d.span) {
                d.L = ell[ks] * tg.stride[ks];
                for (int k = ks - 1; k > kt; --k) {
                    d.Rin *= ell[k];
                    if (ell[k] > 1) {
                        d.frl[nrd] = dev_fastdiv((uint32_t)ell[k]);
                        d.rs[nrd] = tg.stride[k];
                        if (tg.stride[k] & 7) a8 = false;
                        if (tg.stride[k] & 3) a4 = false;
                        ++nrd;
                    }
                }
            }
            d.nrd = nrd;
#ifdef OLAP_TILE_V4
            a8 = false;
#endif
            d.V = a8 ? 8 : (a4 ? 4 : 1);
            np = 1;
            for (int k = 0; k < kt; ++k) {
                d.tlo[k] = lo[k];
                d.tn[k] = ell[k];
            }
            d.tlo[kt] = lo[kt] / tg.ct;
            d.tn[kt] = hi[kt] / tg.ct - d.tlo[kt] + 1;
            for (int k = 0; k <= kt; ++k) {
                np *= d.tn[k];
                d.tfd[k] = dev_fastdiv((uint32_t)d.tn[k]);
            }
            tdesc[q] = d;
            // the summary path's compact descriptor (tile-relative 32-bit geometry)
            SDesc sd;
            memset(&sd, 0, sizeof(sd));
            sd.mode = d.V == 8 && d.nrd <= 1 && !OLAP_TILE_NO_SUMMARY;
            sd.opc = d.opc;
            sd.span = d.span;
            sd.Lin = (int32_t)d.L;
            sd.rad = d.nrd ? (int32_t)d.frl[0].d : 1;
            sd.rs = d.nrd ? (int32_t)d.rs[0] : 0;
            sd.radm = (int32_t)(d.nrd ? d.frl[0].m : dev_fastdiv(1u).m);
            sd.radl = (int32_t)(d.nrd ? d.frl[0].l : dev_fastdiv(1u).l);
            sd.skt = (int32_t)tg.stride[kt];
            sd.lo_kt = (int32_t)d.lo_kt;
            sd.hi_kt = (int32_t)d.hi_kt;
            sd.base_in = (int32_t)d.base_in;
            sd.nkt = kt;
            int64_t ts = 1, jb = d.tlo[kt];
            for (int k = kt - 1; k >= 0; --k) {
                ts *= d.tn[k + 1];
                sd.tstr[k] = (int32_t)ts;
                jb += d.tlo[k] * ts;
            }
            sd.jbase = (int32_t)(-jb);
            // When every run of every pair starts at the same slot of a 32-slot row (run and kt
            // strides multiples of 256 cells), the interior's tree decomposition is the same for all
            // of them: node (rb >> j) + off at level j, rb the run's row start slot.  Precompute it.
            sd.npat = -1;
            if (sd.mode && !d.span && (d.nrd == 0 || (d.rs[0] & 255) == 0) && (tg.stride[kt] & 255) == 0) {
                const uint32_t h0 = (uint32_t)(d.base_in & 7);
                const uint32_t c0 = (uint32_t)(((d.base_in - h0) >> 3) & 31);
                const RunSplit rsp = run_split(h0, (uint32_t)d.L);
                int np2 = 0;
                bool ok = true;
                if (rsp.i0 < rsp.i1) {
                    uint32_t a = c0 + rsp.i0, b = c0 + rsp.i1;
                    auto emit = [&](uint32_t j, uint32_t n) {
                        if (np2 >= 16 || n >= 8192u) ok = false;
                        else sd.pat[np2++] = (uint16_t)(j << 13 | n);
                    };
                    for (uint32_t j = 0; j < (uint32_t)kTreeTop && a < b; ++j) {
                        if (a & 1u) emit(j, a++);
                        if (b & 1u) emit(j, --b);
                        a >>= 1;
                        b >>= 1;
                    }
                    for (; a < b; ++a) emit((uint32_t)kTreeTop, a);
                }
                if (ok) sd.npat = np2;
            }
            sdesc[q] = sd;
        }
        q_pairs[q] = np;
        if (np == 0) {  // identity partials (COUNT, empty, invalid, no owned row: finalize decides)
            psum[q] = 0;
            pext[2 * q] = INT_MIN;
            pext[2 * q + 1] = INT_MIN;
        }
    }
    cells = block_sum<int64_t>(cells, sh);
    if (threadIdx.x == 0 && cells) atomicAdd(totals, (unsigned long long)cells);
}

// Path choice (after the exclusive scan of pair counts -> pair_start[0..nq]).
// ctl: [0] mode (1 = tiles), [1] non-empty tiles, [2] tile pop counter.
// Tiles pay when every staged byte is reused: cells >= 4 x staged cells (staged <= min(pairs,
// ntiles) tiles) and pairs are big enough to amortise their set-up (>= 256 cells each).
// One thread, after the CUB scan (pair_start[nq] = total pairs).
__global__ void tile_scan_kernel(const int64_t* __restrict__ pair_start, int64_t nq, int64_t pairs_cap, TGeo tg,
                                 const unsigned long long* totals, int32_t* ctl, unsigned long long* bytes_acc) {
    const int64_t pairs = pair_start[nq];
    const int64_t cells = (int64_t)totals[0];
    const int64_t staged = min(pairs, tg.ntiles) * tg.tcells;
    const int use = tg.ok && pairs > 0 && pairs <= pairs_cap && cells >= 4 * staged && cells >= 256 * pairs;
    ctl[0] = use;
    ctl[1] = 0;
    ctl[2] = 0;
    if (use) atomicAdd(bytes_acc, (unsigned long long)(cells * 4));
}

// tile id of query d's j-th pair (row-major over its tile box)
__device__ __forceinline__ int64_t pair_tile(const TGeo& tg, const TDesc& d, uint32_t j) {
    int64_t t = 0;
    for (int k = tg.kt; k >= 0; --k) {
        const uint32_t qk = fdiv(j, d.tfd[k]);
        t += (d.tlo[k] + (int64_t)(j - qk * d.tfd[k].d)) * tg.ts[k];
        j = qk;
    }
    return t;
}

// Pairs p0 .. p0+K-1 of the batch: (query, pair index) walked forward from one search.
template <class F>
__device__ __forceinline__ void for_pairs(int64_t nq, const int64_t* __restrict__ pair_start, F&& f) {
    const int64_t total = __ldg(pair_start + nq);
    for (int64_t p0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) * kTilePairsPerThread; p0 < total;
         p0 += (int64_t)gridDim.x * blockDim.x * kTilePairsPerThread) {
        int64_t q = find_query_thread(pair_start, nq, p0);
        int64_t j = p0 - __ldg(pair_start + q), end = __ldg(pair_start + q + 1);
        const int64_t p1 = min(total, p0 + kTilePairsPerThread);
        for (int64_t p = p0; p < p1; ++p) {
            while (p >= end) {  // next query with pairs
                ++q;
                j = 0;
                end = __ldg(pair_start + q + 1);
            }
            f(q, j);
            ++j;
        }
    }
}

// A tile's query list is kept in three op groups (key 3 t + opc - 1: SUM, MIN, MAX) so that
// the consumer warps of a tile mostly run the same specialised loop at the same time (one
// code path in the instruction cache instead of up to 31).
__device__ __forceinline__ int64_t pair_key(const TGeo& tg, const TDesc& d, uint32_t j) {
    return 3 * pair_tile(tg, d, j) + (d.opc - 1);
}

__global__ void tile_count_kernel(TGeo tg, int64_t nq, const int64_t* __restrict__ pair_start,
                                  const TDesc* __restrict__ tdesc, unsigned int* count, const int32_t* ctl) {
    if (!ctl[0]) return;
    for_pairs(nq, pair_start, [&](int64_t q, int64_t j) { atomicAdd(count + pair_key(tg, tdesc[q], (uint32_t)j), 1u); });
}

// non-empty tiles (any order: each is staged once whatever the order)
__global__ void tile_compact_kernel(int64_t ntiles, const unsigned int* __restrict__ tile_start, int32_t* ctl,
                                    uint32_t* nonempty) {
    if (!ctl[0]) return;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < ntiles; t += (int64_t)gridDim.x * blockDim.x)
        if (tile_start[3 * t + 3] > tile_start[3 * t]) nonempty[atomicAdd(ctl + 1, 1)] = (uint32_t)t;
}

// count[] holds the per-tile counts again on entry (it is decremented to 0 here)
__global__ void tile_scatter_kernel(TGeo tg, int64_t nq, const int64_t* __restrict__ pair_start,
                                    const TDesc* __restrict__ tdesc, unsigned int* count,
                                    const unsigned int* __restrict__ tile_start, const int32_t* __restrict__ ctl,
                                    uint32_t* list) {
    if (!ctl[0]) return;
    for_pairs(nq, pair_start, [&](int64_t q, int64_t j) {
        const int64_t k = pair_key(tg, tdesc[q], (uint32_t)j);
        list[tile_start[k] + atomicSub(count + k, 1u) - 1u] = (uint32_t)q;
    });
}

// ------------------------------------------------------------------ reduce

struct TileMeta {
    int64_t t;          // tile id, -1: no more tiles
    int64_t c, ce;      // chunk index along kt and its extent
    int64_t x[kMaxDims];  // tile coordinates of dims < kt
    int32_t x32[kMaxDims];  // the same, 32-bit (summary path: pair index by one warp reduction)
    uint32_t lbeg, cnt;   // the tile's query list
    unsigned int next;    // next list entry to claim
};

// The clipped box of query d in tile (x, c) as a QDesc over the staged tile (cells relative to
// the tile start): runs over dims kt..ks-1, or one span over dim kt.
__device__ __forceinline__ void build_pair_desc(const TGeo& tg, const TDesc& d, int64_t c, int64_t ce, QDesc& pd) {
    // everything inside a staged tile fits 32-bit arithmetic (offsets < kTileCellsMax); no 64-bit
    // division on the common path (column mode needs only the innermost radix, from TDesc)
    const int64_t c0 = c * tg.ct;
    const uint32_t a = (uint32_t)(max(d.lo_kt, c0) - c0), b = (uint32_t)(min(d.hi_kt, c0 + ce - 1) - c0);
    const uint32_t na = b - a + 1;
    const uint32_t skt = (uint32_t)tg.stride[tg.kt];
    const uint32_t base = a * skt + (uint32_t)d.base_in;
    int nrd = d.nrd;
    for (int e = 0; e < nrd; ++e) {
        pd.frl[e] = d.frl[e];
        pd.rs[e] = d.rs[e];
    }
    uint32_t L, R;
    bool radix_na = false;
    if (d.span) {
        L = na * skt;
        R = 1;
    } else {
        L = (uint32_t)d.L;
        R = na * (uint32_t)d.Rin;
        if (na > 1) {
            radix_na = true;
            pd.rs[nrd] = skt;
            ++nrd;
        }
    }
    pd.nrd = nrd;
    const uint32_t V = (uint32_t)d.V, lv = V == 8 ? 3u : (V == 4 ? 2u : 0u);
    const uint32_t h0 = base & (V - 1), nslot = (h0 + L + V - 1) >> lv;
    pd.V = (int32_t)V;
    pd.h0 = (int32_t)h0;
    pd.base_al = base - h0;
    pd.L = L;
    pd.R = R;
    pd.nslot = nslot;
    pd.G = (int64_t)R * nslot;
    pd.vlocal = (int64_t)R * L;
    pd.opc = d.opc;
    pd.tpi = 1;
    pd.shortp = nslot <= (uint32_t)kShortMaxSlots;
    if (OLAP_SM_COLS && pd.shortp && nslot <= 32 && nrd <= 2) return;  // column mode: nothing else needed
    if (OLAP_SM_WIDE && nslot > 32 && nrd <= 2) return;                // wide mode: nothing else needed
    if (radix_na) pd.frl[nrd - 1] = dev_fastdiv(na);
    if (pd.shortp) {
        uint32_t rpt = (uint32_t)kTaskSlots / nslot;
        rpt = rpt < 1 ? 1 : (rpt > 31 ? 31 : rpt);
        pd.T = (int32_t)rpt;
        pd.tasks = (R + rpt - 1) / rpt;
        pd.fni = dev_fastdiv(nslot > 2 ? nslot - 2 : 1u);
        pd.fnslot = dev_fastdiv(1u);
    } else {
        pd.T = nslot < (uint32_t)kTaskSlots ? (int32_t)nslot : kTaskSlots;
        pd.tasks = (pd.G + pd.T - 1) / pd.T;
        pd.fnslot = dev_fastdiv(nslot);
        pd.fni = dev_fastdiv(1u);
    }
}

// Slot trees of a staged tile.  Level 0 holds one entry per 8-cell slot s of the stage buffer (the
// slot's SUM -- float: an fp32 tree of its 8 cells; int32: exact int64 -- its MIN and its MAX);
// level j holds one entry per aligned block of 2^j slots, combined from level j-1 (float SUM: the fp32
// tree continues, so a level-5 entry is an fp32 tree of 256 cells, depth 8, reading R8').  Any slot
// range [a, b) is the union of at most two entries per level (plus whole level-kTreeTop entries):
// a run's interior costs O(log) lookups instead of one per slot.  Each level is stored TRANSPOSED
// over 256-cell rows: node n of level j (row n >> (5 - j), column n mod 2^(5-j)) sits at column x
// kTreeRows + row.  The same node of runs one or more rows apart is then consecutive entries (no
// bank conflicts across lanes walking such runs, and a run-to-run step is a constant address
// increment); kTreeRows is odd so that the columns of one row spread over the banks too.  Written
// by the producer warp once per tile.
template <class Acc> struct TreeGeo;  // slot-tree geometry of the tile size of Acc's dtype (below)
#ifndef OLAP_COL_SLOTS
#define OLAP_COL_SLOTS 6
#endif
constexpr uint32_t kColSlots = OLAP_COL_SLOTS;  // runs of at most this many slots: column mode on raw cells
#ifndef OLAP_PAT_MAX_RUNS
#define OLAP_PAT_MAX_RUNS (1u << 30)
#endif
// pairs of at most this many runs take the per-query pattern (every row-aligned pair by default;
// before the transposed trees, pairs of > 16 runs were walked one run per lane at equal speed)
constexpr uint32_t kPatMaxRuns = OLAP_PAT_MAX_RUNS;
template <class Acc>
struct TreeGeo {
    static constexpr int slots = (int)((tile_cells_max(std::is_same<Acc, AccF>::value) + 7) / 8);
    static constexpr int rows = (slots + 31) / 32 + ((((slots + 31) / 32) & 1) ? 0 : 1);  // odd
    static constexpr int entries = 63 * rows;  // levels 0..5: (32 + 16 + .. + 1) columns of `rows` entries
    // first entry of level j: rows x (32 + 16 + .. + (32 >> (j - 1))) = rows x (64 - (64 >> j))
    __host__ __device__ static constexpr uint32_t lvl_off(int j) { return (uint32_t)rows * (64u - (64u >> j)); }
    // entry index of node n at level j
    __device__ static __forceinline__ uint32_t tidx(int j, uint32_t n) {
        return lvl_off(j) + (n & ((32u >> j) - 1u)) * (uint32_t)rows + (n >> (5 - j));
    }
};
template <class Acc> struct SumEntry;
template <> struct SumEntry<AccF> { using T = float; };
template <> struct SumEntry<AccI> { using T = long long; };
template <class Acc>
constexpr size_t tile_sum_bytes() {  // one stage: sum, min, max trees
    return ((size_t)TreeGeo<Acc>::entries * sizeof(typename SumEntry<Acc>::T) + 2 * (size_t)TreeGeo<Acc>::entries * 4 + 127) &
           ~size_t(127);
}
template <class Acc>
constexpr size_t tile_smem_bytes() {
    return (size_t)kTileStages * (tile_cells_max(std::is_same<Acc, AccF>::value) + kTileSlack) * 4 +
           kTileStages * tile_sum_bytes<Acc>() +
           kTileStages * sizeof(TileMeta) + 3 * kTileStages * sizeof(uint64_t) + 256;
}

template <class Acc>
struct TreeView {
    using ST = typename SumEntry<Acc>::T;
    ST* sum;
    int32_t* mn;
    int32_t* mx;
    __device__ __forceinline__ explicit TreeView(unsigned char* base)
        : sum(reinterpret_cast<ST*>(base)),
          mn(reinterpret_cast<int32_t*>(base + (size_t)TreeGeo<Acc>::entries * sizeof(ST))),
          mx(mn + TreeGeo<Acc>::entries) {}
};

// producer warp: the slot trees of the tile staged in `sb` (cells [0, ncell))
template <typename T, class Acc>
__device__ __forceinline__ void summarize_tile(const uint32_t* __restrict__ sb, uint32_t ncell, unsigned char* base,
                                               int lane) {
    TreeView<Acc> tv(base);
    uint32_t n = (ncell + 7) >> 3;
    // level 0: slot s = lane + 32 it is column lane of row it
    using TG = TreeGeo<Acc>;
    for (uint32_t s = lane, i = lane * (uint32_t)TG::rows; s < n; s += 32, ++i) {
        const uint4 a = *reinterpret_cast<const uint4*>(sb + 8 * s);
        const uint4 b = *reinterpret_cast<const uint4*>(sb + 8 * s + 4);
        const uint32_t v[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
        if constexpr (std::is_same<Acc, AccF>::value) {
            tv.sum[i] = slot_tree<8>(v);
            float mn = __uint_as_float(v[0]), mx = mn;
#pragma unroll
            for (int k = 1; k < 8; ++k) {
                mn = fminf(mn, __uint_as_float(v[k]));
                mx = fmaxf(mx, __uint_as_float(v[k]));
            }
            tv.mn[i] = __float_as_int(mn);
            tv.mx[i] = __float_as_int(mx);
        } else {
            long long t = 0;
            int32_t mn = (int32_t)v[0], mx = mn;
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                t += (int32_t)v[k];
                if (k) {
                    mn = min(mn, (int32_t)v[k]);
                    mx = max(mx, (int32_t)v[k]);
                }
            }
            tv.sum[i] = t;
            tv.mn[i] = mn;
            tv.mx[i] = mx;
        }
    }
#pragma unroll 1
    for (int j = 1; j <= kTreeTop; ++j) {
        __syncwarp();
        n = (n + 1) >> 1;
        for (uint32_t k = lane; k < n; k += 32) {
            // node k = (column c, row r) of level j; its children are columns 2c, 2c + 1 of row r
            const uint32_t c = k & ((32u >> j) - 1u), r = k >> (5 - j);
            const uint32_t d = TG::lvl_off(j) + c * (uint32_t)TG::rows + r;
            const uint32_t c0 = TG::lvl_off(j - 1) + 2 * c * (uint32_t)TG::rows + r, c1 = c0 + (uint32_t)TG::rows;
            if constexpr (std::is_same<Acc, AccF>::value) {
                tv.sum[d] = tv.sum[c0] + tv.sum[c1];
                tv.mn[d] = __float_as_int(fminf(__int_as_float(tv.mn[c0]), __int_as_float(tv.mn[c1])));
                tv.mx[d] = __float_as_int(fmaxf(__int_as_float(tv.mx[c0]), __int_as_float(tv.mx[c1])));
            } else {
                tv.sum[d] = tv.sum[c0] + tv.sum[c1];
                tv.mn[d] = min(tv.mn[c0], tv.mn[c1]);
                tv.mx[d] = max(tv.mx[c0], tv.mx[c1]);
            }
        }
    }
}

// One (query, tile) pair through the slot trees.  The clipped box is R runs of L cells; run r
// starts at cell al + off(r) of the stage (al 32-B aligned, off(r) = (r mod rad) * rs + (r / rad) *
// skt); every run covers slots 0 .. nslot-1 of its own, the first holding cells h0..7, the last
// cells 0..tail-1.
//  * interior slots 1 .. nslot-2: one lane per (run, chunk) -- C = 32 / R chunks per run when the
//    pair has fewer than 32 runs -- decomposes its slot range into tree entries (<= 2 per level);
//  * edge cells (E <= 16 per run): the E needed cells of 32 / E runs per step, one per lane.
// No mask and no idle cell: a lane reads only entries and cells inside the box.
// floor(n / d) for n < 32 (lanes) and 1 <= d <= 32 without a division: n * ceil(2^16 / d) >> 16
// (exact: the rounding excess is below 31 / 2^16 < 1 / d)
__constant__ uint32_t kSmallInv[33] = {0,    65536, 32768, 21846, 16384, 13108, 10923, 9363, 8192, 7282, 6554,
                                        5958, 5462,  5042,  4682,  4370,  4096,  3856,  3641, 3450, 3277, 3121,
                                        2979, 2850,  2731,  2622,  2521,  2428,  2341,  2260, 2185, 2115, 2048};
__device__ __forceinline__ uint32_t small_div(uint32_t n, uint32_t d) { return (n * kSmallInv[d]) >> 16; }


struct RunWalk {  // lane's run cursor: off(r) for r = my, my + g, my + 2g, ...
    uint32_t off, x0, rad, dstep, s0, dcarry;
    __device__ __forceinline__ void init(uint32_t my, uint32_t g, uint32_t rad_, FastDiv fr, uint32_t rs,
                                         uint32_t skt) {
        rad = rad_;
        const uint32_t q = fdiv(my, fr), s1 = fdiv(g, fr);
        x0 = my - q * rad;
        s0 = g - s1 * rad;
        off = x0 * rs + q * skt;
        dstep = s0 * rs + s1 * skt;
        dcarry = skt - rad * rs;
    }
    __device__ __forceinline__ void step() {
        off += dstep;
        x0 += s0;
        if (x0 >= rad) {
            x0 -= rad;
            off += dcarry;
        }
    }
};

template <class Acc, int OPC>
__device__ __forceinline__ void fold_entry(const TreeView<Acc>& tv, uint32_t i, Acc& acc) {
    if constexpr (OPC == OPC_SUM) {
        if constexpr (std::is_same<Acc, AccF>::value) acc.s += (double)tv.sum[i];
        else acc.s += (unsigned long long)tv.sum[i];
    } else if constexpr (OPC == OPC_MIN) {
        if constexpr (std::is_same<Acc, AccF>::value) acc.mn = fminf(acc.mn, __int_as_float(tv.mn[i]));
        else acc.mn = min(acc.mn, tv.mn[i]);
    } else {
        if constexpr (std::is_same<Acc, AccF>::value) acc.mx = fmaxf(acc.mx, __int_as_float(tv.mx[i]));
        else acc.mx = max(acc.mx, tv.mx[i]);
    }
}

// slots [a, b) of the tile through the trees (<= 2 entries per level below kTreeTop)
template <class Acc, int OPC>
__device__ __forceinline__ void fold_range(const TreeView<Acc>& tv, uint32_t a, uint32_t b, Acc& acc) {
#pragma unroll
    for (int j = 0; j < kTreeTop; ++j) {
        if (a >= b) return;
        if (a & 1u) fold_entry<Acc, OPC>(tv, TreeGeo<Acc>::tidx(j, a++), acc);
        if (b & 1u) fold_entry<Acc, OPC>(tv, TreeGeo<Acc>::tidx(j, --b), acc);
        a >>= 1;
        b >>= 1;
    }
    const uint32_t o = TreeGeo<Acc>::lvl_off(kTreeTop);  // one node per row: column 0
    for (; a < b; ++a) fold_entry<Acc, OPC>(tv, o + a, acc);
}

template <typename T, class Acc, int OPC>
__device__ __forceinline__ void pair_summary(const uint32_t* __restrict__ sb, unsigned char* __restrict__ tree,
                                             uint32_t al, uint32_t h0, uint32_t L, uint32_t R, uint32_t rad,
                                             uint32_t na, FastDiv fr, uint32_t rs, uint32_t skt, Acc& acc, int lane) {
    const TreeView<Acc> tv(tree);
    const RunSplit rsp = run_split(h0, L);
    const uint32_t nslot = rsp.nslot;
    const uint32_t ulane = (uint32_t)lane;
    // ---- interior slots through the trees: lane = (run, chunk)
    if (rsp.i0 < rsp.i1) {
        const uint32_t ni = rsp.i1 - rsp.i0;
        // C = 2^lgc chunks per run: the largest power of two with C * min(R, 32) <= 32
        const uint32_t lgc = R >= 32 ? 0u : 31u - __clz(small_div(32u, R));
        const uint32_t C = 1u << lgc;
        const uint32_t g = 32u >> lgc;  // runs per step
        const uint32_t my = ulane >> lgc, ch = ulane & (C - 1u);
        const uint32_t ca = (ni * ch) >> lgc, cb = (ni * (ch + 1u)) >> lgc;  // chunk [ca, cb) of the interior
        RunWalk w;
        w.init(my, g, rad, fr, rs, skt);
        for (uint32_t r0 = 0; r0 < R; r0 += g) {
            if (r0 + my < R) {
                const uint32_t s1 = ((al + w.off) >> 3) + rsp.i0;
                fold_range<Acc, OPC>(tv, s1 + ca, s1 + cb, acc);
            }
            w.step();
        }
    }
    // ---- edge cells: E1 of the first slot (h0 ..), E2 of the last (0 .. tail-1); lanes = (run, cell),
    // g = 32 / E runs per step; kt rows outside, the inner digit inside (offsets advance by g * rs)
    const uint32_t E1 = rsp.E1, E2 = rsp.E2, E = E1 + E2;
    if (E == 0) return;
    const uint32_t g = small_div(32u, E), grp = small_div(ulane, E), e = ulane - grp * E;
    if (grp >= g) return;
    const uint32_t cofs = e < E1 ? h0 + e : 8 * (nslot - 1) + (e - E1);
    auto fold_cell = [&](uint32_t v) {
        if constexpr (OPC == OPC_SUM) {
            if constexpr (std::is_same<Acc, AccF>::value) acc.s += (double)__uint_as_float(v);
            else acc.s += (unsigned long long)(long long)(int32_t)v;
        } else if constexpr (OPC == OPC_MIN) {
            if constexpr (std::is_same<Acc, AccF>::value) acc.mn = fminf(acc.mn, __uint_as_float(v));
            else acc.mn = min(acc.mn, (int32_t)v);
        } else {
            if constexpr (std::is_same<Acc, AccF>::value) acc.mx = fmaxf(acc.mx, __uint_as_float(v));
            else acc.mx = max(acc.mx, (int32_t)v);
        }
    };
    const uint32_t step = g * rs;
    const uint32_t* pk = sb + al + cofs + grp * rs;
    for (uint32_t kr = 0; kr < na; ++kr, pk += skt) {
        const uint32_t* pc = pk;
        uint32_t ri = grp;
        for (; ri + g < rad; ri += 2 * g, pc += 2 * step) {  // two runs per lane in flight
            const uint32_t va = pc[0], vb = pc[step];
            fold_cell(va);
            fold_cell(vb);
        }
        if (ri < rad) fold_cell(pc[0]);
    }
}

// A pair whose runs all start at the same slot of a 32-slot (256-cell) row (SDesc.npat >= 0): the
// interior of every run is the same K tree entries (level j, node (rb >> j) + off, rb = the run's
// row start slot) and the same E edge cells.  One unit = one tree entry or one edge cell of one run;
// lanes = (run group, unit) with U = K + E <= 32 units per run and 32 / U runs per step, every lane
// keeping one unit for the whole pair.  Runs start whole rows apart and the trees are stored
// transposed over rows, so a lane's address advances by a fixed byte step per run (inner digit) and
// per kt row: a step is one load, one fold and one add per lane -- no decomposition, no division,
// no per-load index arithmetic.
template <typename T, class Acc, int OPC>
__device__ __forceinline__ void pair_pattern(const uint32_t* __restrict__ sb, unsigned char* __restrict__ tree,
                                             uint32_t al, uint32_t h0, uint32_t L, uint32_t rad, uint32_t na,
                                             uint32_t rs, uint32_t skt, uint32_t K, uint32_t patw, Acc& acc,
                                             int lane) {
    using ST = typename SumEntry<Acc>::T;
    const RunSplit rsp = run_split(h0, L);
    const uint32_t nslot = rsp.nslot, E1 = rsp.E1, E2 = rsp.E2;
    const uint32_t U = K + E1 + E2;
    const uint32_t ulane = (uint32_t)lane;
    const uint32_t g = small_div(32u, U), grp = small_div(ulane, U), u = ulane - grp * U;
    const uint32_t pw = __shfl_sync(0xffffffffu, patw, (int)(u >> 1) & 7);
    if (na > rad) {  // runs are (kt row, inner digit) pairs either way: split the longer side among the groups
        const uint32_t t = na;
        na = rad;
        rad = t;
        const uint32_t ts = rs;
        rs = skt;
        skt = ts;
    }
    if (grp >= g) return;
    const bool is_tree = u < K;
    constexpr bool wide_sum = std::is_same<Acc, AccI>::value && OPC == OPC_SUM;  // int64 tree entries
    uint32_t addr, step_in, step_kt;  // shared-memory byte address of run (grp, kt row 0) and its steps
    if (is_tree) {
        const uint32_t pt = (u & 1u) ? pw >> 16 : pw & 0xffffu;
        const uint32_t j = pt >> 13, off = pt & 0x1fffu;
        const uint32_t row0 = al >> 8, rsr = rs >> 8, sktr = skt >> 8;  // rows of 256 cells
        const uint32_t idx = TreeGeo<Acc>::lvl_off((int)j) + (off & ((32u >> j) - 1u)) * (uint32_t)TreeGeo<Acc>::rows +
                             (off >> (5 - j)) +
                             row0 + grp * rsr;
        const TreeView<Acc> tv(tree);
        const uint32_t esz = wide_sum ? 8u : 4u;
        addr = smem_addr_u32(OPC == OPC_SUM ? (const void*)tv.sum
                                            : (OPC == OPC_MIN ? (const void*)tv.mn : (const void*)tv.mx)) + idx * esz;
        step_in = g * rsr * esz;
        step_kt = sktr * esz;
    } else {
        const uint32_t e = u - K;
        addr = smem_addr_u32(sb) + 4u * (al + (e < E1 ? h0 + e : 8 * (nslot - 1) + (e - E1)) + grp * rs);
        step_in = 4u * g * rs;
        step_kt = 4u * skt;
    }
    auto fold_one = [&](uint32_t a) {
        if constexpr (wide_sum) {  // tree lanes: 64-bit entry (two 32-bit halves); edge lanes: one cell
            uint32_t lo, hi = 0;
            asm volatile("ld.shared.u32 %0, [%1];" : "=r"(lo) : "r"(a));
            if (is_tree) asm volatile("ld.shared.u32 %0, [%1];" : "=r"(hi) : "r"(a + 4u));
            const long long x = is_tree ? (long long)(((unsigned long long)hi << 32) | lo) : (long long)(int32_t)lo;
            acc.s += (unsigned long long)x;
        } else {
            uint32_t v;
            asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
            if constexpr (OPC == OPC_SUM) acc.s += (double)__uint_as_float(v);
            else if constexpr (OPC == OPC_MIN) {
                if constexpr (std::is_same<Acc, AccF>::value) acc.mn = fminf(acc.mn, __uint_as_float(v));
                else acc.mn = min(acc.mn, (int32_t)v);
            } else {
                if constexpr (std::is_same<Acc, AccF>::value) acc.mx = fmaxf(acc.mx, __uint_as_float(v));
                else acc.mx = max(acc.mx, (int32_t)v);
            }
        }
    };
    (void)sizeof(ST);
    constexpr bool fsum = std::is_same<Acc, AccF>::value && OPC == OPC_SUM;
    for (uint32_t kr = 0; kr < na; ++kr, addr += step_kt) {
        uint32_t a = addr, ri = grp;
        for (; ri + 3 * g < rad; ri += 4 * g, a += 4 * step_in) {  // four runs per lane in flight
            if constexpr (fsum) {
                // float SUM: the four values (tree entries of depth <= 8, or cells) as one fp32 tree of
                // depth 2, then one conversion and one fp64 add (reading R8': fp32 depth <= 10)
                uint32_t v0, v1, v2, v3;
                asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v0) : "r"(a));
                asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v1) : "r"(a + step_in));
                asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v2) : "r"(a + 2 * step_in));
                asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v3) : "r"(a + 3 * step_in));
                acc.s += (double)((__uint_as_float(v0) + __uint_as_float(v1)) +
                                  (__uint_as_float(v2) + __uint_as_float(v3)));
            } else {
                fold_one(a);
                fold_one(a + step_in);
                fold_one(a + 2 * step_in);
                fold_one(a + 3 * step_in);
            }
        }
        for (; ri < rad; ri += g, a += step_in) fold_one(a);
    }
}

template <typename T, class Acc>
__device__ __forceinline__ long long warp_partial(const Acc& acc, int opc) {
    if (opc == OPC_SUM) {
        long long sm = acc.sum_bits();
#pragma unroll
        for (int o = 16; o; o >>= 1) sm = SumOps<Acc>::add(sm, __shfl_xor_sync(0xffffffffu, sm, o));
        return sm;
    }
    if (opc == OPC_MAX) return __reduce_max_sync(0xffffffffu, acc.code_max());
    return __reduce_max_sync(0xffffffffu, ~acc.code_min());
}

template <typename T, class Acc>
__global__ void __launch_bounds__(kTileThreads, 1)
    tile_reduce_kernel(const T* __restrict__ cube, TGeo tg, const TDesc* __restrict__ tdesc,
                       const SDesc* __restrict__ sdesc, const int64_t* __restrict__ pair_start,
                       const unsigned int* __restrict__ tile_start, const uint32_t* __restrict__ nonempty,
                       const uint32_t* __restrict__ list, int32_t* ctl, long long* __restrict__ partial,
                       QDesc* __restrict__ pds_g) {
    if (!*(volatile int32_t*)ctl) return;
    extern __shared__ __align__(128) unsigned char smem[];
    constexpr int64_t kCells = tile_cells_max(std::is_same<Acc, AccF>::value);
    constexpr size_t kBufBytes = (size_t)(kCells + kTileSlack) * 4;
    uint32_t* buf = reinterpret_cast<uint32_t*>(smem);  // kTileStages x (kCells + kTileSlack) cells
    unsigned char* sums = smem + kTileStages * kBufBytes;  // kTileStages x tile_sum_bytes
    TileMeta* meta = reinterpret_cast<TileMeta*>(sums + kTileStages * tile_sum_bytes<Acc>());
    uint64_t* full = reinterpret_cast<uint64_t*>(meta + kTileStages);
    uint64_t* empty = full + kTileStages;
    uint64_t* ready = empty + kTileStages;
    // the general-geometry fallback's per-warp descriptors live in global memory (L1-resident):
    // shared memory holds two 64-KiB float stages with their trees and nothing else fits
    QDesc* pds = pds_g + (size_t)blockIdx.x * kTileConsumers;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    if (threadIdx.x == 0) {
        for (int s = 0; s < kTileStages; ++s) {
            mbar_init(full + s, 1);
            mbar_init(empty + s, kTileConsumers);
            mbar_init(ready + s, 32);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const int64_t bufcells = kCells + kTileSlack;
    if (w == 0) {
        // producer warp: pop a non-empty tile, stage it with bulk copies (lane 0), wait for it to
        // land, write its slot summaries (all lanes), then release it to the consumers (ready)
        const uint32_t nne = (uint32_t)ctl[1];
        const int kt = tg.kt;
        for (int64_t i = 0;; ++i) {
            const int s = (int)(i % kTileStages);
            const uint32_t ph = (uint32_t)((i / kTileStages) & 1);
            if (i >= kTileStages) mbar_wait_sleep(empty + s, ph ^ 1u);
            TileMeta& m = meta[s];
            uint32_t k = 0;
            if (lane == 0) {
                k = (uint32_t)atomicAdd(ctl + 2, 1);
                if (k >= nne) {
                    m.t = -1;
                } else {
                    const int64_t t = nonempty[k];
                    m.t = t;
                    m.next = 0;
                    m.lbeg = tile_start[3 * t];
                    m.cnt = tile_start[3 * t + 3] - m.lbeg;
                    int64_t r = t;
                    m.c = r % tg.nct;
                    r /= tg.nct;
                    int64_t start = m.c * tg.ct * tg.stride[kt];
                    for (int e = kt - 1; e >= 0; --e) {
                        const int64_t xe = r % tg.ext[e];
                        r /= tg.ext[e];
                        m.x[e] = xe;
                        m.x32[e] = (int32_t)xe;
                        start += xe * tg.stride[e];
                    }
                    m.ce = min(tg.ct, tg.ext[kt] - m.c * tg.ct);
                    const int64_t cells = (m.ce * tg.stride[kt] + 3) & ~3ll;
                    const uint32_t bytes = (uint32_t)(cells * 4);
                    mbar_arrive_tx(full + s, bytes);
                    const char* src = reinterpret_cast<const char*>(cube + start);
                    char* dst = reinterpret_cast<char*>(buf + s * bufcells);
                    for (uint32_t o = 0; o < bytes; o += 16384u)
                        bulk_g2s(dst + o, src + o, min(16384u, bytes - o), full + s);
                }
            }
            k = __shfl_sync(0xffffffffu, k, 0);
            if (k >= nne) {
                mbar_arrive(ready + s);  // every lane: the end-of-tiles marker is visible
                break;
            }
            mbar_wait(full + s, ph);
            const uint32_t ncell = (uint32_t)(m.ce * tg.stride[kt]);
            summarize_tile<T, Acc>(buf + s * bufcells, ncell, sums + s * tile_sum_bytes<Acc>(), lane);
            mbar_arrive(ready + s);  // release: this lane's summaries (and lane 0's meta) before the consumers
        }
        return;
    }
    // consumers: every pair of the staged tile, one warp per pair
    QDesc& pd = pds[w - 1];
    for (int64_t i = 0;; ++i) {
        const int s = (int)(i % kTileStages);
        const uint32_t ph = (uint32_t)((i / kTileStages) & 1);
        mbar_wait(ready + s, ph);
        TileMeta& m = meta[s];
        const int64_t t = m.t;
        if (t < 0) break;  // the end-of-tiles marker has no copy behind it: never wait on full[s] for it
        // also observe the bulk copy's own completion (already complete: the producer waited for it
        // before summarising) -- a direct acquire of the async-proxy writes, not only through ready[s]
#ifndef OLAP_NO_FULL_WAIT
        mbar_wait(full + s, ph);
#endif
        const uint32_t* sb = buf + s * bufcells;
        unsigned char* sm = sums + s * tile_sum_bytes<Acc>();
        const uint32_t c0 = (uint32_t)(m.c * tg.ct), ce = (uint32_t)m.ce;
        for (;;) {
            uint32_t e = 0;
            if (lane == 0) e = atomicAdd(&m.next, 1u);
            e = __shfl_sync(0xffffffffu, e, 0);
            if (e >= m.cnt) break;
            const int64_t q = __ldg(list + m.lbeg + e);
            // the query's compact descriptor: words 0-15 by four uniform (broadcast) 16-B loads, the
            // tile-box strides (words 16..) by lane k < nkt
            const int4* sd4 = reinterpret_cast<const int4*>(sdesc + q);
            // every load of the pair's set-up issued at once (one global latency, not three in a row)
            const int4 w0 = __ldg(sd4), w1 = __ldg(sd4 + 1), w2 = __ldg(sd4 + 2), w3 = __ldg(sd4 + 3);
            const int32_t tw = __ldg(reinterpret_cast<const int32_t*>(sdesc + q) + 16 + (lane & 7));
            const uint32_t patw = (uint32_t)__ldg(reinterpret_cast<const int32_t*>(sdesc + q) + 24 + (lane & 7));
            const int64_t ps = __ldg(pair_start + q);
            const int mode = w0.x;
            long long v;
            int opc;
            int64_t p;
            if (mode) {
                opc = w0.y;
                const uint32_t span = (uint32_t)w0.z, Lin = (uint32_t)w0.w, rad = (uint32_t)w1.x;
                const uint32_t rs = (uint32_t)w1.y, skt = (uint32_t)w1.z, lo_kt = (uint32_t)w1.w;
                const uint32_t hi_kt = (uint32_t)w2.x, base_in = (uint32_t)w2.y;
                const int32_t jbase = w2.z;
                FastDiv fr;
                fr.d = rad;
                fr.m = (uint32_t)w2.w;
                fr.l = (uint32_t)w3.x;
                const int nkt = w3.y;
                // pair index j of this tile in the query's tile box (one warp reduction)
                const int32_t tj = lane < nkt ? m.x32[lane] * tw : 0;
                const int32_t j = jbase + (int32_t)m.c + __reduce_add_sync(0xffffffffu, tj);
                p = ps + j;
                // the query's box clipped to this tile's chunk [c0, c0 + ce) of dim kt
                const uint32_t a = max(lo_kt, c0) - c0, b = min(hi_kt, c0 + ce - 1) - c0, na = b - a + 1;
                const uint32_t base = a * skt + base_in;
                const uint32_t L = span ? na * skt : Lin, R = span ? 1u : na * rad;
                const uint32_t h0 = base & 7u, al = base - h0;
                Acc acc;
                acc.init();
                if (((h0 + L + 7) >> 3) <= kColSlots) {
                    // short runs (<= kColSlots = 6 slots): column mode over the raw cells, 5+ runs per step
                    QDesc qd;
                    qd.nslot = (h0 + L + 7) >> 3;
                    qd.R = R;
                    qd.base_al = al;
                    qd.h0 = (int32_t)h0;
                    qd.L = L;
                    qd.rs[0] = rs;
                    qd.rs[1] = skt;
                    qd.frl[0] = fr;
                    if (opc == OPC_SUM) stream_cols<Acc, OPC_SUM, 8, 2>(sb, qd, acc, lane);
                    else if (opc == OPC_MIN) stream_cols<Acc, OPC_MIN, 8, 2>(sb, qd, acc, lane);
                    else stream_cols<Acc, OPC_MAX, 8, 2>(sb, qd, acc, lane);
                } else if (w3.z >= 0 && !span && R <= kPatMaxRuns &&
                           (uint32_t)w3.z + run_split(h0, L).E1 + run_split(h0, L).E2 <= 32u) {
                    // row-aligned runs: the precomputed per-query pattern, one unit per lane
                    const uint32_t K = (uint32_t)w3.z;
                    if (opc == OPC_SUM) pair_pattern<T, Acc, OPC_SUM>(sb, sm, al, h0, L, rad, na, rs, skt, K, patw, acc, lane);
                    else if (opc == OPC_MIN) pair_pattern<T, Acc, OPC_MIN>(sb, sm, al, h0, L, rad, na, rs, skt, K, patw, acc, lane);
                    else pair_pattern<T, Acc, OPC_MAX>(sb, sm, al, h0, L, rad, na, rs, skt, K, patw, acc, lane);
                } else if (opc == OPC_SUM) {
                    pair_summary<T, Acc, OPC_SUM>(sb, sm, al, h0, L, R, span ? 1u : rad, span ? 1u : na, fr, rs, skt, acc, lane);
                } else if (opc == OPC_MIN) {
                    pair_summary<T, Acc, OPC_MIN>(sb, sm, al, h0, L, R, span ? 1u : rad, span ? 1u : na, fr, rs, skt, acc, lane);
                } else {
                    pair_summary<T, Acc, OPC_MAX>(sb, sm, al, h0, L, R, span ? 1u : rad, span ? 1u : na, fr, rs, skt, acc, lane);
                }
                v = warp_partial<T, Acc>(acc, opc);
            } else {  // general geometry: the item path's streamers over the staged tile
                const TDesc& d = tdesc[q];
                if (lane == 0) build_pair_desc(tg, d, m.c, m.ce, pd);
                int64_t jj = 0;
                for (int k = 0; k < tg.kt; ++k) jj = jj * d.tn[k] + (m.x[k] - d.tlo[k]);
                jj = jj * d.tn[tg.kt] + (m.c - d.tlo[tg.kt]);
                p = ps + jj;
                __syncwarp();
                Acc acc;
                acc.init();
                stream_item<T, Acc, true>(reinterpret_cast<const T*>(sb), pd, 0, pd.tasks, acc, lane, 0, 1);
                opc = pd.opc;
                v = warp_partial<T, Acc>(acc, opc);
            }
            if (lane == 0) partial[p] = v;
            __syncwarp();
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(empty + s);
    }
}

// One block per query with pairs: fold its pair partials in pair order (fixed tree) into the
// per-query partial format (sum, max code, ~min code).
template <class Acc>
__global__ void __launch_bounds__(256) pair_fold_kernel(int64_t nq, const int64_t* __restrict__ pair_start,
                                                        const TDesc* __restrict__ tdesc, const int32_t* ctl,
                                                        const long long* __restrict__ partial, int64_t* psum,
                                                        int32_t* pext) {
    if (!ctl[0]) return;
    __shared__ long long sh[8];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int64_t q = blockIdx.x; q < nq; q += gridDim.x) {
        const int64_t b = __ldg(pair_start + q), e = __ldg(pair_start + q + 1);
        if (b == e) continue;  // identity partials written by tile_desc_kernel
        const int opc = tdesc[q].opc;
        long long v = opc == OPC_SUM ? 0ll : (long long)INT_MIN;
        for (int64_t p = b + threadIdx.x; p < e; p += blockDim.x) {
            const long long x = __ldcg(partial + p);
            v = opc == OPC_SUM ? SumOps<Acc>::add(v, x) : max(v, x);
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) {
            const long long y = __shfl_xor_sync(0xffffffffu, v, o);
            v = opc == OPC_SUM ? SumOps<Acc>::add(v, y) : max(v, y);
        }
        if (lane == 0) sh[w] = v;
        __syncthreads();
        if (threadIdx.x == 0) {
            long long f = sh[0];
            for (int i = 1; i < 8; ++i) f = opc == OPC_SUM ? SumOps<Acc>::add(f, sh[i]) : max(f, sh[i]);
            psum[q] = opc == OPC_SUM ? f : 0;
            pext[2 * q] = opc == OPC_MAX ? (int32_t)f : INT_MIN;
            pext[2 * q + 1] = opc == OPC_MIN ? (int32_t)f : INT_MIN;
        }
        __syncthreads();
    }
}
