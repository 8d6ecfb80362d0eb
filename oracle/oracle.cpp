/*
 * oracle/oracle.cpp — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU implementation of what the OLAP hot path
 * computes (Malik, Riha, Shea, El-Ghazawi, IPDPSW 2012; /root/reference/PAPER.md).
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference legs may load this library.  It shares no code, header, table or
 * helper with the CUDA path under paper_conf_ipps_malikrse12_b200/, and it
 * includes nothing from include/.
 *
 * What it computes (each function cites the passage it follows):
 *   oracle_query      — sub-cube ("area of limited search") aggregation of a
 *                       query Q(C_1(f_1,t_1),...,C_N(f_N,t_N))        Eq. 1
 *                       over the box f_i..t_i (inclusive), box volume Eq. 3 PAPER.md:136-141 (corrected,
 *                       DESIGN.md reading R1/R2), aggregates "count, sum, average,
 *                       maximum etc."                                    PAPER.md:25 (reading R4: + MIN)
 *                       Plain odometer over the box in row-major order.  PAPER.md:109-112, Fig. 2 :151
 *   oracle_dict_*     — one text-to-integer dictionary per text column  PAPER.md:252-256 (§III-F)
 *                       as std::map<std::string,int32_t>; id = rank in byte order (reading R11).
 *   oracle_tablescan  — the paper's GPU query Q_D over a column-store fact table
 *                       (Eq. 11-12): conditions on dimension
 *                       columns, aggregate of one data column, COUNT = matching rows.
 *   oracle_rollup / oracle_convert_range — the multi-resolution cube set
 *                       (Fig. 1, Eq. 1-2): coarse cells
 *                       aggregate the fine cells mapping to them; a level-r range in
 *                       level-R members.
 *   oracle_factbuild  — the cube built from fact rows ("the GPU performs ... building the
 *                       cube from relational tables"): every row adds its
 *                       measure (or 1) into the cell its dimension ids name.  Plain row
 *                       loop; int32 wraps mod 2^32; float32 adds each cell's values in row
 *                       order in double and rounds once into the cell (reading R27).
 *   oracle_factscan   — filtered aggregation over a fact table of translated
 *                       (integer) dimension columns and one data column  PAPER.md:206-208 (§III-E)
 *                       used as an independent path to the cube answer for SUM.
 *   oracle_gen_*      — the counter-based synthetic cell generator (splitmix64),
 *                       re-implemented here independently of the CUDA fill kernel
 *                       (both sides implement the same formula).
 *
 * Accumulation (readings R7/R8): int32 cells sum into uint64 with two's-complement
 * wraparound and are reported as int64; float32 cells sum in double in row-major
 * order; MIN/MAX compare with '<' in the cell type; COUNT is the box volume V;
 * AVG = (double)SUM / (double)V.  An empty box (lo>hi in any dimension) yields
 * flags=1 with COUNT=SUM=0 (reading R10).
 *
 * Parity pins for every function live in tests/test_oracle_*.py (-m "not gpu").
 */
#include <climits>
#include <cstdint>
#include <cstring>
#include <map>
#include <string>
#include <vector>
#include <chrono>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {

constexpr int ORC_INT32 = 1;
constexpr int ORC_FLOAT32 = 2;

constexpr int ORC_SUM = 0, ORC_COUNT = 1, ORC_MIN = 2, ORC_MAX = 3, ORC_AVG = 4;

constexpr int ORC_GEN_UNIFORM = 1;  // counter-hash uniform
constexpr int ORC_GEN_AFFINE = 2;   // v(x) = c0 + sum_d c_d x_d

struct Range { int64_t lo, hi; };
struct Result { int64_t i; double d; uint32_t flags; uint32_t pad; };

/* splitmix64 of (seed, index): the counter-based generator of DESIGN.md "inputs". */
uint64_t splitmix64_at(uint64_t seed, uint64_t idx) {
    uint64_t z = seed + (idx + 1ull) * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

/* A cube the oracle can read: either a host array or a procedural generator. */
struct Cube {
    int nd;
    int64_t n[8];
    int dtype;
    const void* cells;      // row-major, unpadded; nullptr => procedural
    int gen;
    uint64_t seed;
    double params[9];       // affine: c0, c_1..c_N

    /* value of the cell with linear row-major index idx and coordinates x */
    int32_t cell_i32(int64_t idx, const int64_t* x) const {
        if (cells) return static_cast<const int32_t*>(cells)[idx];
        if (gen == ORC_GEN_UNIFORM) {
            uint64_t z = splitmix64_at(seed, (uint64_t)idx);
            return (int32_t)(z >> 43) - (1 << 20);           // uniform in [-2^20, 2^20)
        }
        double v = params[0];
        for (int d = 0; d < nd; ++d) v += params[1 + d] * (double)x[d];
        return (int32_t)v;
    }
    float cell_f32(int64_t idx, const int64_t* x) const {
        if (cells) return static_cast<const float*>(cells)[idx];
        if (gen == ORC_GEN_UNIFORM) {
            uint64_t z = splitmix64_at(seed, (uint64_t)idx);
            return (float)(z >> 40) * (1.0f / 16777216.0f);   // k * 2^-24, k in [0, 2^24)
        }
        double v = params[0];
        for (int d = 0; d < nd; ++d) v += params[1 + d] * (double)x[d];
        return (float)v;
    }
};

/* Eq. 1 query over the box lo..hi (inclusive) — the plain definition, odometer order. */
int query_one(const Cube& c, const Range* r, int op, Result* out) {
    std::memset(out, 0, sizeof(*out));
    for (int d = 0; d < c.nd; ++d)
        if (r[d].lo < 0 || r[d].hi >= c.n[d]) return -2;          // out of bounds
    if (op < ORC_SUM || op > ORC_AVG) return -1;
    for (int d = 0; d < c.nd; ++d)
        if (r[d].lo > r[d].hi) { out->flags = 1; return 0; }       // empty box (R10)

    /* Eq. 3 (corrected): V = prod (t_i - f_i + 1) */
    __int128 V = 1;
    for (int d = 0; d < c.nd; ++d) V *= (__int128)(r[d].hi - r[d].lo + 1);
    if (V > (__int128)INT64_MAX) return -1;

    if (op == ORC_COUNT) { out->i = (int64_t)V; return 0; }        // COUNT = V (R5), reads no cell

    int64_t s[8];
    s[c.nd - 1] = 1;
    for (int d = c.nd - 2; d >= 0; --d) s[d] = s[d + 1] * c.n[d + 1];

    int64_t x[8];
    for (int d = 0; d < c.nd; ++d) x[d] = r[d].lo;

    uint64_t sum_u = 0; double sum_f = 0.0;
    int32_t mn_i = INT32_MAX, mx_i = INT32_MIN;
    float mn_f = 0.f, mx_f = 0.f;
    int64_t cnt = 0;
    for (;;) {
        int64_t idx = 0;
        for (int d = 0; d < c.nd; ++d) idx += x[d] * s[d];
        if (c.dtype == ORC_INT32) {
            int32_t v = c.cell_i32(idx, x);
            sum_u += (uint64_t)(int64_t)v;
            if (v < mn_i) mn_i = v;
            if (mx_i < v) mx_i = v;
        } else {
            float v = c.cell_f32(idx, x);
            sum_f += (double)v;
            if (cnt == 0) { mn_f = v; mx_f = v; }
            if (v < mn_f) mn_f = v;
            if (mx_f < v) mx_f = v;
        }
        ++cnt;
        int d = c.nd - 1;                                           // advance innermost with carry
        while (d >= 0) {
            if (++x[d] <= r[d].hi) break;
            x[d] = r[d].lo;
            --d;
        }
        if (d < 0) break;
    }
    if ((__int128)cnt != V) return -1;                               // loop counter must equal V

    if (c.dtype == ORC_INT32) {
        int64_t sum = (int64_t)sum_u;
        switch (op) {
            case ORC_SUM: out->i = sum; break;
            case ORC_MIN: out->i = mn_i; break;
            case ORC_MAX: out->i = mx_i; break;
            case ORC_AVG: out->d = (double)sum / (double)V; break;
        }
    } else {
        out->i = 0;
        switch (op) {
            case ORC_SUM: out->d = sum_f; break;
            case ORC_MIN: out->d = (double)mn_f; break;
            case ORC_MAX: out->d = (double)mx_f; break;
            case ORC_AVG: out->d = sum_f / (double)V; break;
        }
    }
    return 0;
}

int make_cube(Cube* c, int nd, const int64_t* extents, int dtype, const void* cells,
              int gen, uint64_t seed, const double* params) {
    if (nd < 1 || nd > 8) return -1;
    if (dtype != ORC_INT32 && dtype != ORC_FLOAT32) return -1;
    std::memset(c, 0, sizeof(*c));
    c->nd = nd;
    c->dtype = dtype;
    for (int d = 0; d < nd; ++d) {
        if (extents[d] < 1) return -1;
        c->n[d] = extents[d];
    }
    c->cells = cells;
    c->gen = gen;
    c->seed = seed;
    if (!cells) {
        if (gen != ORC_GEN_UNIFORM && gen != ORC_GEN_AFFINE) return -1;
        if (gen == ORC_GEN_AFFINE)
            for (int d = 0; d <= nd; ++d) c->params[d] = params[d];
    }
    return 0;
}

/* ---- dictionary: one std::map per text column ---- */
struct Dict {
    std::map<std::string, int32_t> m;
    std::vector<std::string> inv;
};

}  // namespace

extern "C" {

uint64_t oracle_splitmix64(uint64_t seed, uint64_t idx) { return splitmix64_at(seed, idx); }

/* Materialise ncells cells of a procedural cube (row-major) — for cross-checks. */
int oracle_fill(int nd, const int64_t* extents, int dtype, int gen, uint64_t seed,
                const double* params, int64_t first, int64_t ncells, void* out) {
    Cube c;
    if (make_cube(&c, nd, extents, dtype, nullptr, gen, seed, params)) return -1;
    int64_t x[8];
    for (int64_t k = 0; k < ncells; ++k) {
        int64_t idx = first + k, rem = idx;
        for (int d = nd - 1; d >= 0; --d) { x[d] = rem % c.n[d]; rem /= c.n[d]; }
        if (dtype == ORC_INT32) static_cast<int32_t*>(out)[k] = c.cell_i32(idx, x);
        else static_cast<float*>(out)[k] = c.cell_f32(idx, x);
    }
    return 0;
}

/*
 * Answer nq queries (ranges: nq*nd, query-major) on a host cube (cells != NULL)
 * or a procedural one (cells == NULL: gen/seed/params).  nthreads > 1 runs an
 * OpenMP loop over queries (the paper's OpenMP partition),
 * used only to time the baseline.  Returns 0, or -2 on the first out-of-bounds
 * query (bad_query set), -1 on invalid arguments.
 */
int oracle_query(int nd, const int64_t* extents, int dtype, const void* cells,
                 int gen, uint64_t seed, const double* params,
                 int64_t nq, const void* ranges, const int32_t* ops, void* results,
                 int nthreads, int64_t* bad_query) {
    Cube c;
    if (make_cube(&c, nd, extents, dtype, cells, gen, seed, params)) return -1;
    const Range* r = static_cast<const Range*>(ranges);
    Result* out = static_cast<Result*>(results);
    int64_t first_bad = -1;
    int status = 0;
    if (nthreads <= 1) {
        for (int64_t q = 0; q < nq; ++q) {
            int st = query_one(c, r + q * nd, ops[q], out + q);
            if (st) { status = st; first_bad = q; break; }
        }
    } else {
#ifdef _OPENMP
        std::vector<int> st(nq, 0);
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
        for (int64_t q = 0; q < nq; ++q) st[q] = query_one(c, r + q * nd, ops[q], out + q);
        for (int64_t q = 0; q < nq; ++q)
            if (st[q]) { status = st[q]; first_bad = q; break; }
#else
        return -1;
#endif
    }
    if (bad_query) *bad_query = first_bad;
    return status;
}

int oracle_max_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* ---- dictionaries ---- */
void* oracle_dict_build(const char* bytes, const int64_t* offsets, int64_t n) {
    Dict* d = new Dict();
    for (int64_t i = 0; i < n; ++i)
        d->m.emplace(std::string(bytes + offsets[i], (size_t)(offsets[i + 1] - offsets[i])), 0);
    int32_t id = 0;
    for (auto& kv : d->m) { kv.second = id++; d->inv.push_back(kv.first); }
    return d;
}

int64_t oracle_dict_size(void* h) { return (int64_t)static_cast<Dict*>(h)->m.size(); }

/* ids[i] = dict[key i] or -1 if absent; returns the number of misses */
int64_t oracle_dict_translate(void* h, const char* bytes, const int64_t* offsets, int64_t n,
                              int32_t* ids) {
    Dict* d = static_cast<Dict*>(h);
    int64_t miss = 0;
    for (int64_t i = 0; i < n; ++i) {
        auto it = d->m.find(std::string(bytes + offsets[i], (size_t)(offsets[i + 1] - offsets[i])));
        if (it == d->m.end()) { ids[i] = -1; ++miss; }
        else ids[i] = it->second;
    }
    return miss;
}

/* first id whose key is >= s (upper=0) or > s (upper=1); D if none — string ranges (reading R11) */
int64_t oracle_dict_bound(void* h, const char* s, int64_t len, int upper) {
    Dict* d = static_cast<Dict*>(h);
    std::string k(s, (size_t)len);
    auto it = upper ? d->m.upper_bound(k) : d->m.lower_bound(k);
    return it == d->m.end() ? (int64_t)d->m.size() : (int64_t)it->second;
}

int oracle_dict_lookup(void* h, int32_t id, const char** bytes, int64_t* len) {
    Dict* d = static_cast<Dict*>(h);
    if (id < 0 || (size_t)id >= d->inv.size()) return -1;
    *bytes = d->inv[id].data();
    *len = (int64_t)d->inv[id].size();
    return 0;
}

void oracle_dict_destroy(void* h) { delete static_cast<Dict*>(h); }

/*
 * Fact-table scan: rows r in [0,nrows) with ndims integer
 * dimension columns dims[d*nrows + r] (already translated to ids) and one data
 * column.  For each query (ranges nd per query, inclusive), aggregate the data
 * column over rows whose every dimension value lies in its range.  Only SUM and
 * the fact COUNT are reported: out_sum[q] (int64 for int32 data, else the
 * double's bits), out_count[q].
 */
int oracle_factscan(int64_t nrows, int nd, const int32_t* dims, int dtype, const void* data,
                    int64_t nq, const void* ranges, int64_t* out_sum, int64_t* out_count) {
    const Range* r = static_cast<const Range*>(ranges);
    for (int64_t q = 0; q < nq; ++q) {
        const Range* rq = r + q * nd;
        uint64_t su = 0; double sf = 0.0; int64_t cnt = 0;
        for (int64_t row = 0; row < nrows; ++row) {
            bool hit = true;
            for (int d = 0; d < nd && hit; ++d) {
                int64_t v = dims[(int64_t)d * nrows + row];
                hit = (rq[d].lo <= v && v <= rq[d].hi);
            }
            if (!hit) continue;
            ++cnt;
            if (dtype == ORC_INT32) su += (uint64_t)(int64_t)static_cast<const int32_t*>(data)[row];
            else sf += (double)static_cast<const float*>(data)[row];
        }
        if (dtype == ORC_INT32) out_sum[q] = (int64_t)su;
        else std::memcpy(&out_sum[q], &sf, sizeof(double));
        out_count[q] = cnt;
    }
    return 0;
}

/*
 * Cube build from fact rows (§III-F: the text columns are
 * already integer ids).  ids[d*nrows + r] is row r's member id in dimension d; a row with
 * an id outside [0, n_d) adds nothing.  vals (nrows cells of the cube's dtype) or NULL to
 * add 1 per row.  cells: the row-major host cube, updated in place:
 *   int32:   cell += v (mod 2^32) row by row;
 *   float32: acc[cell] = sum of the cell's values in row order, in double; then
 *            cell = (float)((double)cell + acc[cell]) once (reading R27).
 */
int oracle_factbuild(int nd, const int64_t* extents, int dtype, int64_t nrows, const int32_t* ids,
                     const void* vals, void* cells) {
    int64_t ncells = 1;
    for (int d = 0; d < nd; ++d) ncells *= extents[d];
    std::vector<double> acc(dtype == ORC_FLOAT32 ? ncells : 0, 0.0);
    std::vector<char> touched(dtype == ORC_FLOAT32 ? ncells : 0, 0);
    for (int64_t r = 0; r < nrows; ++r) {
        int64_t idx = 0;
        bool ok = true;
        for (int d = 0; d < nd; ++d) {
            const int64_t x = ids[(int64_t)d * nrows + r];
            if (x < 0 || x >= extents[d]) ok = false;
            idx = idx * extents[d] + x;
        }
        if (!ok) continue;
        if (dtype == ORC_INT32) {
            int32_t* c = static_cast<int32_t*>(cells);
            const uint32_t v = vals ? (uint32_t)static_cast<const int32_t*>(vals)[r] : 1u;
            c[idx] = (int32_t)((uint32_t)c[idx] + v);
        } else {
            acc[idx] += vals ? (double)static_cast<const float*>(vals)[r] : 1.0;
            touched[idx] = 1;
        }
    }
    if (dtype == ORC_FLOAT32) {
        float* c = static_cast<float*>(cells);
        for (int64_t i = 0; i < ncells; ++i)
            if (touched[i]) c[i] = (float)((double)c[i] + acc[i]);
    }
    return 0;
}

/*
 * Fact-table query Q_D (Eq. 11; §III-E): the table
 * is a set of columns ("all columns of the table one after another"), dimension columns
 * hold integer member ids (one column per dimension x level), data columns hold the
 * measures.  Query q has conditions conds[cond_off[q] .. cond_off[q+1]) — each a column
 * and an inclusive range [f, t] on its ids — a data column and an aggregate op.  A row
 * matches when it satisfies every condition; the answer aggregates the data column over
 * matching rows.  COUNT counts matching rows (facts).  AVG = SUM / COUNT.  No matching
 * row: flags = 1 (EMPTY), i = d = 0.  Accumulation as oracle_query (readings R7/R8).
 * cols[c] points to nrows 4-byte values; dtypes[c] is ORC_INT32 or ORC_FLOAT32.
 */
struct TCond { int32_t col; int32_t pad; int64_t lo, hi; };

int oracle_tablescan(int64_t nrows, int ncols, const void* const* cols, const int32_t* dtypes, int64_t nq,
                     const int64_t* cond_off, const void* conds_v, const int32_t* data_cols, const int32_t* ops,
                     void* results, int nthreads) {
    const TCond* conds = static_cast<const TCond*>(conds_v);
    Result* out = static_cast<Result*>(results);
    for (int64_t q = 0; q < nq; ++q) {
        if (data_cols[q] < 0 || data_cols[q] >= ncols || ops[q] < ORC_SUM || ops[q] > ORC_AVG) return -1;
        for (int64_t k = cond_off[q]; k < cond_off[q + 1]; ++k)
            if (conds[k].col < 0 || conds[k].col >= ncols || dtypes[conds[k].col] != ORC_INT32) return -1;
    }
#ifdef _OPENMP
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads > 1 ? nthreads : 1)
#endif
    for (int64_t q = 0; q < nq; ++q) {
        const int dc = data_cols[q];
        const bool fl = dtypes[dc] == ORC_FLOAT32;
        uint64_t su = 0;
        double sf = 0.0;
        int64_t cnt = 0;
        int32_t mn_i = INT32_MAX, mx_i = INT32_MIN;
        float mn_f = 0.f, mx_f = 0.f;
        for (int64_t r = 0; r < nrows; ++r) {
            bool hit = true;
            for (int64_t k = cond_off[q]; k < cond_off[q + 1] && hit; ++k) {
                const int64_t v = static_cast<const int32_t*>(cols[conds[k].col])[r];
                hit = conds[k].lo <= v && v <= conds[k].hi;
            }
            if (!hit) continue;
            if (fl) {
                const float v = static_cast<const float*>(cols[dc])[r];
                sf += (double)v;
                if (cnt == 0) { mn_f = v; mx_f = v; }
                if (v < mn_f) mn_f = v;
                if (mx_f < v) mx_f = v;
            } else {
                const int32_t v = static_cast<const int32_t*>(cols[dc])[r];
                su += (uint64_t)(int64_t)v;
                if (v < mn_i) mn_i = v;
                if (mx_i < v) mx_i = v;
            }
            ++cnt;
        }
        Result res;
        std::memset(&res, 0, sizeof(res));
        if (cnt == 0) {
            res.flags = 1;
        } else {
            const int op = ops[q];
            if (op == ORC_COUNT) res.i = cnt;
            else if (!fl) {
                const int64_t sum = (int64_t)su;
                if (op == ORC_SUM) res.i = sum;
                else if (op == ORC_MIN) res.i = mn_i;
                else if (op == ORC_MAX) res.i = mx_i;
                else res.d = (double)sum / (double)cnt;
            } else {
                if (op == ORC_SUM) res.d = sf;
                else if (op == ORC_MIN) res.d = (double)mn_f;
                else if (op == ORC_MAX) res.d = (double)mx_f;
                else res.d = sf / (double)cnt;
            }
        }
        out[q] = res;
    }
    return 0;
}

/*
 * Multi-resolution cube set (Fig. 1, Eq. 1-2).  Dimension d
 * has levels 0 (coarsest) .. L-1 (finest); level_ids[d*L + r][x] is the level-r member
 * of finest member x.
 *
 * oracle_rollup: the cell of a cube at level rc is the aggregate (op: SUM, MIN or MAX)
 * of every cell of the level-rf cube (rf > rc) whose members map to it.  Plain loop over
 * the fine cells; int32 SUM wraps mod 2^32 into the int32 cell, float32 SUM accumulates
 * in double and rounds once to float32.  fine/coarse: row-major host arrays.
 */
int oracle_rollup(int nd, int L, const int64_t* n_finest, const int32_t* const* level_ids, int dtype,
                  int rf, const int64_t* ext_f, const void* fine, int rc, const int64_t* ext_c, void* coarse, int op) {
    (void)L;
    int64_t nf = 1, ncc = 1;
    for (int d = 0; d < nd; ++d) { nf *= ext_f[d]; ncc *= ext_c[d]; }
    // member map level rf -> level rc per dimension, through any finest member
    std::vector<std::vector<int64_t>> up(nd);
    for (int d = 0; d < nd; ++d) {
        up[d].assign(ext_f[d], -1);
        for (int64_t x = 0; x < n_finest[d]; ++x)
            up[d][level_ids[d * L + rf][x]] = level_ids[d * L + rc][x];
    }
    std::vector<double> accf(ncc, 0.0);
    std::vector<int64_t> acci(ncc, 0);
    std::vector<char> seen(ncc, 0);
    std::vector<int64_t> x(nd, 0);
    for (int64_t i = 0; i < nf; ++i) {
        int64_t rem = i, ci = 0, mul = 1;
        for (int d = nd - 1; d >= 0; --d) { x[d] = rem % ext_f[d]; rem /= ext_f[d]; }
        for (int d = nd - 1; d >= 0; --d) { ci += up[d][x[d]] * mul; mul *= ext_c[d]; }
        if (dtype == ORC_INT32) {
            const int64_t v = static_cast<const int32_t*>(fine)[i];
            if (op == ORC_SUM) acci[ci] += v;
            else if (!seen[ci] || (op == ORC_MIN ? v < acci[ci] : v > acci[ci])) acci[ci] = v;
        } else {
            const double v = static_cast<const float*>(fine)[i];
            if (op == ORC_SUM) accf[ci] += v;
            else if (!seen[ci] || (op == ORC_MIN ? v < accf[ci] : v > accf[ci])) accf[ci] = v;
        }
        seen[ci] = 1;
    }
    for (int64_t c = 0; c < ncc; ++c) {
        if (dtype == ORC_INT32) static_cast<int32_t*>(coarse)[c] = (int32_t)(uint32_t)(uint64_t)acci[c];
        else static_cast<float*>(coarse)[c] = (float)accf[c];
    }
    return 0;
}

/* Eq. 1 condition [f, t] given at level r, expressed at level R >= r: every level-R member
 * whose level-r ancestor lies in [f, t] (scan of the finest members). */
int oracle_convert_range(int L, int64_t n_finest, const int32_t* const* ids_of_dim, int r, int R, int64_t f,
                         int64_t t, int64_t* out_lo, int64_t* out_hi) {
    (void)L;
    int64_t lo = INT64_MAX, hi = INT64_MIN;
    for (int64_t x = 0; x < n_finest; ++x) {
        const int64_t a = ids_of_dim[r][x];
        if (a < f || a > t) continue;
        const int64_t b = ids_of_dim[R][x];
        if (b < lo) lo = b;
        if (b > hi) hi = b;
    }
    if (lo > hi) { lo = 1; hi = 0; }
    *out_lo = lo;
    *out_hi = hi;
    return 0;
}

}  // extern "C"
