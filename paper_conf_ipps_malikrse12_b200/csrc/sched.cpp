// sched.cpp — the dispatcher: Fig. 10's scheduling algorithm
// over partitions whose performance functions follow Eq. 4
// (PAPER.md:161-164).  Host code: the decision per query is a handful of flops, so it
// belongs next to the launches it drives, not on the GPU.
//
// Readings (R19-R25):
//   R19 an idle queue is free at the query's arrival: T_Q <- max(T_Q, T_O);
//   R20 a partition stays busy until the query's response time: T_Q <- T_R (the paper's
//       T_Q + T_GPU whenever translation does not delay the start);
//   R22 step 5 compares processing times (T_CPU vs the fastest GPU partition's T_GPU);
//       if P_BD holds only cube partitions that lose that comparison, the earliest
//       response among them is taken (Fig. 10 leaves this case open);
//   R23 step 6's min |T_D - T_R| with P_BD empty is the earliest response, ties to the
//       lowest index;
//   R24 P_BD = { i : T_D - T_R,i > 0 } (strict);
//   R25 Eq. 4's ranges: x < x_split -> range A, else range B (Eq. 7 / 10 use "<").
#include <cmath>
#include <mutex>
#include <new>
#include <vector>

#include "olap.h"

namespace olap {
int set_error(int status, const char* fmt, ...);
void clear_error();
}  // namespace olap

struct olap_sched {
    std::vector<olap_sched_partition> parts;
    std::vector<double> t_q;  // T_Q per partition
    double t_q_trans = 0.0;   // T_Q|TRANS
    double t_c = 0.0;
    std::mutex mu;
};

namespace {

double eval_perf(const olap_perf_fn& f, double x) {
    return x < f.x_split ? f.a1 * std::pow(x, f.p1) + f.b1 : f.a2 * std::pow(x, f.p2) + f.b2;
}

void decide(olap_sched* s, const olap_sched_query& q, olap_sched_decision& d) {
    const int np = (int)s->parts.size();
    const double inf = HUGE_VAL;
    const double t_o = q.t_arrival;
    const double t_d = t_o + s->t_c;  // step 1
    for (int i = 0; i < np; ++i) s->t_q[i] = std::fmax(s->t_q[i], t_o);  // R19
    s->t_q_trans = std::fmax(s->t_q_trans, t_o);
    // steps 2-3: processing and response time on every partition
    double t_proc[64], t_r[64];
    bool in_bd[64];
    double fastest_table = inf;
    bool any_bd = false;
    for (int i = 0; i < np; ++i) {
        const olap_sched_partition& p = s->parts[i];
        const double x = p.kind == OLAP_PART_CUBE ? q.cube_mb : q.col_frac;
        t_proc[i] = x >= 0.0 ? eval_perf(p.perf, x) : inf;
        if (t_proc[i] == inf) t_r[i] = inf;
        else if (p.needs_translation && q.t_trans > 0.0)
            t_r[i] = std::fmax(s->t_q[i], s->t_q_trans + q.t_trans) + t_proc[i];
        else t_r[i] = s->t_q[i] + t_proc[i];
        in_bd[i] = t_d - t_r[i] > 0.0;  // step 4 (R24)
        any_bd = any_bd || in_bd[i];
        if (p.kind == OLAP_PART_TABLE && t_proc[i] < fastest_table) fastest_table = t_proc[i];
    }
    int c = -1;
    if (any_bd) {
        // step 5: a cube partition in P_BD faster than the fastest table partition ...
        for (int i = 0; i < np && c < 0; ++i)
            if (in_bd[i] && s->parts[i].kind == OLAP_PART_CUBE && t_proc[i] < fastest_table) c = i;
        // ... else the slowest table partition in P_BD (first in FOR-loop order) ...
        for (int i = 0; i < np && c < 0; ++i)
            if (in_bd[i] && s->parts[i].kind == OLAP_PART_TABLE) c = i;
        // ... else (only slower cube partitions meet T_D) the earliest response among them (R22)
        if (c < 0)
            for (int i = 0; i < np; ++i)
                if (in_bd[i] && (c < 0 || t_r[i] < t_r[c])) c = i;
    } else {
        // step 6: nobody meets T_D — the earliest response (R23)
        double best = inf;
        for (int i = 0; i < np; ++i)
            if (t_r[i] < best) {
                best = t_r[i];
                c = i;
            }
    }
    d.t_deadline = t_d;
    if (c < 0) {
        d.partition = -1;
        d.translated = 0;
        d.t_response = inf;
        d.t_est = inf;
        return;
    }
    d.partition = c;
    d.translated = (s->parts[c].needs_translation && q.t_trans > 0.0) ? 1 : 0;
    if (d.translated) s->t_q_trans = s->t_q_trans + q.t_trans;
    s->t_q[c] = t_r[c];  // R20
    d.t_response = t_r[c];
    d.t_est = t_proc[c];
}

bool finite_or_inf(double v) { return !std::isnan(v); }

}  // namespace

extern "C" {

int olap_sched_create(int nparts, const olap_sched_partition* parts, double t_c, olap_sched** out) {
    olap::clear_error();
    if (!out || !parts) return olap::set_error(OLAP_E_INVALID, "olap_sched_create: NULL argument");
    if (nparts < 1 || nparts > 64) return olap::set_error(OLAP_E_INVALID, "nparts %d not in [1,64]", nparts);
    if (!(t_c > 0.0)) return olap::set_error(OLAP_E_INVALID, "T_C must be > 0");
    for (int i = 0; i < nparts; ++i) {
        const olap_sched_partition& p = parts[i];
        if (p.kind != OLAP_PART_CUBE && p.kind != OLAP_PART_TABLE)
            return olap::set_error(OLAP_E_INVALID, "partition %d: kind %d", i, p.kind);
        const olap_perf_fn& f = p.perf;
        const double v[7] = {f.x_split, f.a1, f.p1, f.b1, f.a2, f.p2, f.b2};
        for (double x : v)
            if (!finite_or_inf(x)) return olap::set_error(OLAP_E_INVALID, "partition %d: NaN in perf", i);
    }
    olap_sched* s = new (std::nothrow) olap_sched();
    if (!s) return olap::set_error(OLAP_E_NOMEM, "host allocation failed");
    s->parts.assign(parts, parts + nparts);
    s->t_q.assign(nparts, 0.0);
    s->t_c = t_c;
    *out = s;
    return OLAP_OK;
}

int olap_sched_submit(olap_sched* s, int64_t n, const olap_sched_query* qs, olap_sched_decision* out) {
    olap::clear_error();
    if (!s) return olap::set_error(OLAP_E_INVALID, "scheduler handle is NULL");
    if (n < 0) return olap::set_error(OLAP_E_INVALID, "n < 0");
    if (n == 0) return OLAP_OK;
    if (!qs || !out) return olap::set_error(OLAP_E_INVALID, "NULL buffer");
    for (int64_t k = 0; k < n; ++k)
        if (std::isnan(qs[k].t_arrival) || std::isnan(qs[k].cube_mb) || std::isnan(qs[k].col_frac) ||
            !(qs[k].t_trans >= 0.0))
            return olap::set_error(OLAP_E_INVALID, "query %lld: NaN or negative T_TRANS", (long long)k);
    std::lock_guard<std::mutex> lk(s->mu);
    for (int64_t k = 0; k < n; ++k) decide(s, qs[k], out[k]);
    return OLAP_OK;
}

int olap_sched_complete(olap_sched* s, int partition, double t_est, double t_real) {
    olap::clear_error();
    if (!s) return olap::set_error(OLAP_E_INVALID, "scheduler handle is NULL");
    if (partition < 0 || partition >= (int)s->parts.size())
        return olap::set_error(OLAP_E_INVALID, "partition %d out of range", partition);
    if (!std::isfinite(t_est) || !std::isfinite(t_real))
        return olap::set_error(OLAP_E_INVALID, "non-finite time");
    std::lock_guard<std::mutex> lk(s->mu);
    s->t_q[partition] = s->t_q[partition] + (t_real - t_est);
    return OLAP_OK;
}

int olap_sched_queues(const olap_sched* s, double* t_q) {
    olap::clear_error();
    if (!s || !t_q) return olap::set_error(OLAP_E_INVALID, "NULL argument");
    for (size_t i = 0; i < s->t_q.size(); ++i) t_q[i] = s->t_q[i];
    t_q[s->t_q.size()] = s->t_q_trans;
    return OLAP_OK;
}

int olap_sched_destroy(olap_sched* s) {
    olap::clear_error();
    delete s;
    return OLAP_OK;
}

}  // extern "C"
