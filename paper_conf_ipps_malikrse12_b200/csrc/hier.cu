// hier.cu — multi-resolution cube set.
//
// "One OLAP system can have multiple pre-calculated cubes with different resolutions
// ... years (low resolution), months, days, hours (high resolution) ... it is always
// desirable to respond to the query using a cube with lowest possible resolution"
// (Fig. 1).  A condition of Eq. 1 carries its resolution r
// and the query needs the cube of resolution R = max r_i (Eq. 2,
// PAPER.md:132-136).
//
// olap_hier: per dimension, levels 0 (coarsest) .. L-1 (finest); every level-r member
//   is a contiguous block of finest members (non-decreasing level ids).
// olap_cube_rollup: builds the level-rc cube from a level-rf cube on the GPU — one
//   thread per coarse cell aggregates the fine cells of its preimage box in row-major
//   order (SUM in int64 / fp64, MIN, MAX), so results match the plain definition.
// olap_cubeset_query: Eq. 2 routing.  A query goes to the cube of resolution exactly R;
//   SUM, which roll-up preserves, may also use the lowest-resolution finer cube; with no
//   usable cube the query is flagged OLAP_RESULT_INVALID (answer it from the fact table,
//   olap_table_*, as the paper does on the GPU).
#include <algorithm>
#include <climits>
#include <cstring>
#include <new>
#include <vector>

#include "common.cuh"

struct olap_hier {
    int nd = 0, L = 0;
    std::vector<int64_t> n_finest;
    // starts[d][r][m] = first finest member of level-r member m; starts[d][r][n_r] = n_finest
    std::vector<std::vector<std::vector<int64_t>>> starts;
    // ids[d][r][x] = level-r member of finest member x
    std::vector<std::vector<std::vector<int32_t>>> ids;
    int64_t extent(int d, int r) const { return (int64_t)starts[d][r].size() - 1; }
};

struct olap_cubeset {
    const olap_hier* h = nullptr;
    std::vector<olap_cube*> cube;  // per level (borrowed)
};

extern "C" int olap_cube_info(const olap_cube* c, int64_t* local_rows, int64_t* local_cells, void** d_cells);
extern "C" int olap_query_batch(olap_cube* c, int64_t nq, const olap_range* ranges, const int32_t* ops,
                                olap_result* results);

namespace olap {

int cube_geometry(const olap_cube* c, int* nd, int64_t* n, int* dtype, int64_t* pitch, int64_t* nshards);
int cube_layout(const olap_cube* c);

constexpr int kMaxHierDims = 8;

struct RollArgs {
    int nd;
    int dtype, op;
    int64_t cext[kMaxHierDims];    // coarse extents
    int64_t cstride[kMaxHierDims]; // coarse strides (cells, padded pitch)
    int64_t fstride[kMaxHierDims]; // fine strides
    const int64_t* pre[kMaxHierDims];  // per dim: preimage start (level rf) of every coarse member, + sentinel
};

template <typename T>
__global__ void rollup_kernel(const T* __restrict__ fine, T* __restrict__ coarse, RollArgs a, int64_t ncoarse) {
    for (int64_t ci = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; ci < ncoarse;
         ci += (int64_t)gridDim.x * blockDim.x) {
        // coordinates of the coarse cell (logical, row-major)
        int64_t rem = ci, cm[kMaxHierDims], lo[kMaxHierDims], hi[kMaxHierDims];
        for (int d = a.nd - 1; d >= 0; --d) {
            cm[d] = rem % a.cext[d];
            rem /= a.cext[d];
        }
        int64_t coff = 0, base = 0;
        for (int d = 0; d < a.nd; ++d) {
            coff += cm[d] * a.cstride[d];
            lo[d] = a.pre[d][cm[d]];
            hi[d] = a.pre[d][cm[d] + 1] - 1;
            base += lo[d] * a.fstride[d];
        }
        // odometer over the preimage box, innermost fastest (row-major order)
        int64_t x[kMaxHierDims];
        for (int d = 0; d < a.nd; ++d) x[d] = lo[d];
        long long si = 0;
        double sf = 0.0;
        T ext = fine[base];
        int64_t off = base;
        for (;;) {
            const T v = fine[off];
            if (a.op == OLAP_SUM) {
                if (sizeof(T) == 4 && a.dtype == OLAP_INT32) si += (long long)v;
                else sf += (double)v;
            } else if (a.op == OLAP_MIN) {
                ext = v < ext ? v : ext;
            } else {
                ext = ext < v ? v : ext;
            }
            int d = a.nd - 1;
            while (d >= 0) {
                if (++x[d] <= hi[d]) {
                    off += a.fstride[d];
                    break;
                }
                off -= (x[d] - 1 - lo[d]) * a.fstride[d];
                x[d] = lo[d];
                --d;
            }
            if (d < 0) break;
        }
        if (a.op == OLAP_SUM) {
            if (a.dtype == OLAP_INT32) coarse[coff] = (T)(int32_t)(uint32_t)(unsigned long long)si;
            else coarse[coff] = (T)sf;
        } else {
            coarse[coff] = ext;
        }
    }
}

}  // namespace olap

using namespace olap;

extern "C" {

int olap_hier_create(int ndims, int nlevels, const int64_t* n_finest, const int32_t* const* level_ids, olap_hier** out) {
    clear_error();
    if (!out || !n_finest || !level_ids) return set_error(OLAP_E_INVALID, "olap_hier_create: NULL argument");
    if (ndims < 1 || ndims > kMaxHierDims || nlevels < 1 || nlevels > 16)
        return set_error(OLAP_E_INVALID, "ndims %d / nlevels %d out of range", ndims, nlevels);
    olap_hier* h = new (std::nothrow) olap_hier();
    if (!h) return set_error(OLAP_E_NOMEM, "host allocation failed");
    h->nd = ndims;
    h->L = nlevels;
    h->n_finest.assign(n_finest, n_finest + ndims);
    h->starts.resize(ndims);
    h->ids.resize(ndims);
    for (int d = 0; d < ndims; ++d) {
        const int64_t n = n_finest[d];
        if (n < 1) {
            delete h;
            return set_error(OLAP_E_INVALID, "dimension %d: n_finest < 1", d);
        }
        h->starts[d].resize(nlevels);
        h->ids[d].resize(nlevels);
        for (int r = 0; r < nlevels; ++r) {
            const int32_t* a = level_ids[d * nlevels + r];
            if (!a) {
                delete h;
                return set_error(OLAP_E_INVALID, "dimension %d level %d: NULL ids", d, r);
            }
            h->ids[d][r].assign(a, a + n);
            std::vector<int64_t>& st = h->starts[d][r];
            for (int64_t x = 0; x < n; ++x) {
                const int32_t prev = x ? a[x - 1] : -1;
                if (a[x] != prev && a[x] != prev + 1) {
                    delete h;
                    return set_error(OLAP_E_INVALID, "dimension %d level %d: ids must start at 0 and be "
                                     "non-decreasing by steps of 0/1 (member %lld)", d, r, (long long)x);
                }
                if (a[x] != prev) st.push_back(x);
                if (r == nlevels - 1 && a[x] != x) {
                    delete h;
                    return set_error(OLAP_E_INVALID, "dimension %d: the finest level must be the identity", d);
                }
                // a member of level r must lie inside one member of every coarser level
                if (r > 0 && x > 0 && a[x] == prev && h->ids[d][r - 1][x] != h->ids[d][r - 1][x - 1]) {
                    delete h;
                    return set_error(OLAP_E_INVALID, "dimension %d: level %d member splits a level %d member", d,
                                     r, r - 1);
                }
            }
            st.push_back(n);
        }
    }
    *out = h;
    return OLAP_OK;
}

int olap_hier_extents(const olap_hier* h, int level, int64_t* extents) {
    clear_error();
    if (!h || !extents || level < 0 || level >= h->L) return set_error(OLAP_E_INVALID, "bad hierarchy / level");
    for (int d = 0; d < h->nd; ++d) extents[d] = h->extent(d, level);
    return OLAP_OK;
}

int olap_hier_destroy(olap_hier* h) {
    clear_error();
    delete h;
    return OLAP_OK;
}

// Eq. 1 conditions [f, t] at levels r_i -> [lo, hi] at level `target` (>= every r_i):
// the first / last target member inside f / t (a coarse member is a contiguous block).
int olap_hier_convert(const olap_hier* h, int64_t nq, const olap_range* ranges, const int32_t* levels, int target,
                      olap_range* out) {
    clear_error();
    if (!h || nq < 0 || (nq && (!ranges || !levels || !out))) return set_error(OLAP_E_INVALID, "NULL argument");
    if (target < 0 || target >= h->L) return set_error(OLAP_E_INVALID, "target level %d", target);
    for (int64_t q = 0; q < nq; ++q) {
        for (int d = 0; d < h->nd; ++d) {
            const int64_t c = q * h->nd + d;
            const int r = levels[c];
            if (r < 0 || r > target)
                return set_error(OLAP_E_INVALID, "query %lld dimension %d: level %d not in [0,%d]", (long long)q, d,
                                 r, target);
            const olap_range g = ranges[c];
            if (g.lo < 0 || g.hi >= h->extent(d, r))
                return set_error(OLAP_E_RANGE, "query %lld dimension %d: [%lld,%lld] outside level %d's [0,%lld)",
                                 (long long)q, d, (long long)g.lo, (long long)g.hi, r, (long long)h->extent(d, r));
            olap_range o;
            if (g.lo > g.hi) {
                o.lo = 1;
                o.hi = 0;
            } else {
                const std::vector<int64_t>& st = h->starts[d][r];
                const std::vector<int32_t>& to = h->ids[d][target];
                o.lo = to[st[g.lo]];
                o.hi = to[st[g.hi + 1] - 1];
            }
            out[c] = o;
        }
    }
    return OLAP_OK;
}

int olap_cube_rollup(const olap_hier* h, const olap_cube* fine, int fine_level, olap_cube* coarse, int coarse_level,
                     int op) {
    clear_error();
    if (!h || !fine || !coarse) return set_error(OLAP_E_INVALID, "NULL argument");
    if (op != OLAP_SUM && op != OLAP_MIN && op != OLAP_MAX) return set_error(OLAP_E_INVALID, "roll-up op %d", op);
    if (fine_level < 0 || fine_level >= h->L || coarse_level < 0 || coarse_level > fine_level)
        return set_error(OLAP_E_INVALID, "levels fine %d coarse %d", fine_level, coarse_level);
    int ndf, ndc, dtf, dtc;
    int64_t nf[8], nc[8], pf, pc, sf, sc;
    cube_geometry(fine, &ndf, nf, &dtf, &pf, &sf);
    cube_geometry(coarse, &ndc, nc, &dtc, &pc, &sc);
    if (ndf != h->nd || ndc != h->nd || dtf != dtc) return set_error(OLAP_E_INVALID, "cube dims / dtype mismatch");
    if (sf != 1 || sc != 1) return set_error(OLAP_E_UNSUPPORTED, "roll-up needs unsharded cubes");
    if (cube_layout(fine) != OLAP_LAYOUT_ROWMAJOR || cube_layout(coarse) != OLAP_LAYOUT_ROWMAJOR)
        return set_error(OLAP_E_UNSUPPORTED, "roll-up needs row-major cubes");
    for (int d = 0; d < h->nd; ++d)
        if (nf[d] != h->extent(d, fine_level) || nc[d] != h->extent(d, coarse_level))
            return set_error(OLAP_E_INVALID, "dimension %d: cube extents do not match the hierarchy levels", d);
    RollArgs a;
    std::memset(&a, 0, sizeof(a));
    a.nd = h->nd;
    a.dtype = dtf;
    a.op = op;
    std::vector<int64_t*> dev;
    int rc = OLAP_OK;
    for (int d = h->nd - 1; d >= 0; --d) {
        a.cext[d] = nc[d];
        a.cstride[d] = d == h->nd - 1 ? 1 : a.cstride[d + 1] * (d == h->nd - 2 ? pc : nc[d + 1]);
        a.fstride[d] = d == h->nd - 1 ? 1 : a.fstride[d + 1] * (d == h->nd - 2 ? pf : nf[d + 1]);
    }
    void *dfine, *dcoarse;
    olap_cube_info(fine, nullptr, nullptr, &dfine);
    olap_cube_info(coarse, nullptr, nullptr, &dcoarse);
    for (int d = 0; d < h->nd; ++d) {
        // preimage of coarse member m at the fine level: [id_f(start_c[m]), id_f(start_c[m+1]-1)]
        std::vector<int64_t> pre(nc[d] + 1);
        const std::vector<int64_t>& st = h->starts[d][coarse_level];
        for (int64_t m = 0; m <= nc[d]; ++m)
            pre[m] = m < nc[d] ? h->ids[d][fine_level][st[m]] : nf[d];
        int64_t* p = nullptr;
        if (cudaMalloc(&p, sizeof(int64_t) * pre.size()) != cudaSuccess ||
            cudaMemcpy(p, pre.data(), sizeof(int64_t) * pre.size(), cudaMemcpyHostToDevice) != cudaSuccess) {
            rc = set_error(OLAP_E_CUDA, "roll-up map upload failed");
            cudaFree(p);
            break;
        }
        dev.push_back(p);
        a.pre[d] = p;
    }
    if (rc == OLAP_OK) {
        int64_t ncoarse = 1;
        for (int d = 0; d < h->nd; ++d) ncoarse *= nc[d];
        const int grid = (int)std::min<int64_t>((ncoarse + 255) / 256, 148 * 16);
        if (dtf == OLAP_INT32)
            rollup_kernel<int32_t><<<grid, 256>>>(static_cast<const int32_t*>(dfine), static_cast<int32_t*>(dcoarse), a,
                                                  ncoarse);
        else
            rollup_kernel<float><<<grid, 256>>>(static_cast<const float*>(dfine), static_cast<float*>(dcoarse), a,
                                                ncoarse);
        cudaError_t e = cudaGetLastError();
        if (e == cudaSuccess) e = cudaDeviceSynchronize();
        if (e != cudaSuccess) rc = set_error(OLAP_E_CUDA, "rollup_kernel: %s", cudaGetErrorString(e));
    }
    for (auto p : dev) cudaFree(p);
    return rc;
}

int olap_cubeset_create(const olap_hier* h, olap_cubeset** out) {
    clear_error();
    if (!h || !out) return set_error(OLAP_E_INVALID, "NULL argument");
    olap_cubeset* s = new (std::nothrow) olap_cubeset();
    if (!s) return set_error(OLAP_E_NOMEM, "host allocation failed");
    s->h = h;
    s->cube.assign(h->L, nullptr);
    *out = s;
    return OLAP_OK;
}

int olap_cubeset_add(olap_cubeset* s, int level, olap_cube* c) {
    clear_error();
    if (!s || !c || level < 0 || level >= s->h->L) return set_error(OLAP_E_INVALID, "bad cube set / level");
    int nd, dt;
    int64_t n[8], pitch, ns;
    cube_geometry(c, &nd, n, &dt, &pitch, &ns);
    if (nd != s->h->nd || ns != 1) return set_error(OLAP_E_INVALID, "cube does not match the hierarchy (or sharded)");
    for (int d = 0; d < nd; ++d)
        if (n[d] != s->h->extent(d, level))
            return set_error(OLAP_E_INVALID, "dimension %d: extent %lld != level %d size %lld", d, (long long)n[d],
                             level, (long long)s->h->extent(d, level));
    s->cube[level] = c;
    return OLAP_OK;
}

int olap_cubeset_destroy(olap_cubeset* s) {
    clear_error();
    delete s;
    return OLAP_OK;
}

int olap_cubeset_query(olap_cubeset* s, int64_t nq, const olap_range* ranges, const int32_t* levels, const int32_t* ops,
                       olap_result* results, int32_t* level_used) {
    clear_error();
    if (!s) return set_error(OLAP_E_INVALID, "cube set is NULL");
    if (nq < 0) return set_error(OLAP_E_INVALID, "nq < 0");
    if (nq == 0) return OLAP_OK;
    if (!ranges || !levels || !ops || !results) return set_error(OLAP_E_INVALID, "NULL buffer");
    const int nd = s->h->nd, L = s->h->L;
    std::vector<int32_t> target(nq, -1);
    for (int64_t q = 0; q < nq; ++q) {
        int R = 0;  // Eq. 2: R = max r_i
        for (int d = 0; d < nd; ++d) {
            const int r = levels[q * nd + d];
            if (r < 0 || r >= L)
                return set_error(OLAP_E_INVALID, "query %lld dimension %d: level %d", (long long)q, d, r);
            R = std::max(R, r);
        }
        if (s->cube[R]) target[q] = R;
        else if (ops[q] == OLAP_SUM)  // roll-up preserves sums: any finer cube answers exactly
            for (int r = R + 1; r < L; ++r)
                if (s->cube[r]) {
                    target[q] = r;
                    break;
                }
    }
    for (int R = 0; R < L; ++R) {
        std::vector<int64_t> qs;
        for (int64_t q = 0; q < nq; ++q)
            if (target[q] == R) qs.push_back(q);
        if (qs.empty()) continue;
        std::vector<olap_range> rin(qs.size() * nd), rout(qs.size() * nd);
        std::vector<int32_t> lv(qs.size() * nd), op(qs.size());
        for (size_t i = 0; i < qs.size(); ++i) {
            for (int d = 0; d < nd; ++d) {
                rin[i * nd + d] = ranges[qs[i] * nd + d];
                lv[i * nd + d] = levels[qs[i] * nd + d];
            }
            op[i] = ops[qs[i]];
        }
        int rc = olap_hier_convert(s->h, (int64_t)qs.size(), rin.data(), lv.data(), R, rout.data());
        if (rc) return rc;
        std::vector<olap_result> res(qs.size());
        rc = olap_query_batch(s->cube[R], (int64_t)qs.size(), rout.data(), op.data(), res.data());
        if (rc) return rc;
        for (size_t i = 0; i < qs.size(); ++i) results[qs[i]] = res[i];
    }
    for (int64_t q = 0; q < nq; ++q) {
        if (target[q] < 0) {
            olap_result r;
            std::memset(&r, 0, sizeof(r));
            r.flags = OLAP_RESULT_INVALID;
            results[q] = r;
        }
        if (level_used) level_used[q] = target[q];
    }
    return OLAP_OK;
}

}  // extern "C"
