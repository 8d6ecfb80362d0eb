"""oracle.sched — TEST INFRASTRUCTURE ONLY (same rules as the rest of oracle/).

The paper's scheduling algorithm, Fig. 10 (§III-G,
PAPER.md:274-320), written out step by step in plain Python, with its performance
functions:
  - Eq. 4 — a piecewise estimate over two size ranges;
  - Eq. 7 / Eq. 10 — the CPU cube model, T = a * SC^p (+ b);
  - Eq. 13-15 — the GPU fact-table model, T = a * (C/C_TOT) + b;
  - Eq. 17-18 — the translation bound.
The correction after Fig. 10 is also here: the real processing
time minus the estimate is added to the queue's T_Q.

B200 reading (DESIGN.md §8(f) NEXT #4, readings R19-R25):
  - A partition is either a CUBE partition (the paper's CPU partition: it answers
    from pre-computed cubes, estimate x = SC_size in MB, Eq. 3) or a TABLE partition
    (the paper's GPU partitions: they scan the fact table, estimate x = C_QD/C_TOTAL,
    Eq. 12-13).
  - Each partition carries its own performance function. This replaces the paper's
    index map j = [i/2] (S17).
  - Each partition has a flag for whether its queries must pass through the
    translation queue. The paper sets it for the GPU partitions only.

Every step below is numbered as in Fig. 10.  Nothing here is shared with the
product library (paper_conf_ipps_malikrse12_b200/csrc/sched.cu).
"""
from __future__ import annotations

import math

CUBE, TABLE = 0, 1
INF = math.inf


def perf(fn, x):
    """Eq. 4: f_A on range A (x < x_split), f_B on range B (R25); each f = a * x^p + b
    (Eq. 5-10 use p != 1 with b = 0 on range A and p = 1 on range B; Eq. 14-15 are p = 1)."""
    split, a1, p1, b1, a2, p2, b2 = fn
    if x < split:
        return a1 * math.pow(x, p1) + b1
    return a2 * math.pow(x, p2) + b2


def trans_upper_bound(dict_lengths, t_per_entry=0.0138e-6):
    """Eq. 17-18: ceil(T_TRANS) = sum over the query's text conditions of P_DICT(D_L|i),
    P_DICT(D_L) = 0.0138e-6 * D_L on the paper's test system."""
    t = 0.0
    for dl in dict_lengths:
        t += t_per_entry * dl
    return t


class Fig10:
    """One scheduler instance: partitions = [(kind, needs_translation, perf_fn)] in the
    order Fig. 10's FOR loop visits them (slow -> fast), t_c = T_C."""

    def __init__(self, partitions, t_c):
        self.parts = list(partitions)
        self.t_c = t_c
        self.t_q = [0.0] * len(self.parts)  # T_Q|C, T_Q|G1..G6
        self.t_q_trans = 0.0                # T_Q|TRANS

    def submit(self, t_o, cube_x, table_x, t_trans):
        """One query Q. cube_x = SC_size in MB (< 0: no cube answers Q); table_x = C_QD/C_TOT
        (< 0: no table answers Q); t_trans = T_TRANS (0: no text parameters).
        Returns (partition, translated, T_R, T_D, T_est); partition -1 if nothing can answer."""
        # 1.) deadline
        t_d = t_o + self.t_c
        # R19: a queue that has drained is free at T_O (a query cannot start before it arrives)
        for i in range(len(self.parts)):
            if self.t_q[i] < t_o:
                self.t_q[i] = t_o
        if self.t_q_trans < t_o:
            self.t_q_trans = t_o
        # 2.) processing time on every partition
        t_proc = []
        for kind, _, fn in self.parts:
            x = cube_x if kind == CUBE else table_x
            t_proc.append(perf(fn, x) if x >= 0 else INF)
        # 3.) response time on every partition (translation first where the partition needs it)
        t_r = []
        for i, (kind, needs_trans, _) in enumerate(self.parts):
            if t_proc[i] == INF:
                t_r.append(INF)
            elif needs_trans and t_trans > 0:
                t_r.append(max(self.t_q[i], self.t_q_trans + t_trans) + t_proc[i])
            else:
                t_r.append(self.t_q[i] + t_proc[i])
        # 4.) P_BD: partitions that answer before the deadline, (T_D - T_R) > 0  (R24)
        p_bd = [i for i in range(len(self.parts)) if t_d - t_r[i] > 0]
        chosen = -1
        if p_bd:
            # 5.) a CUBE partition in P_BD that is faster than the fastest TABLE partition (R22)
            fastest_table = INF
            for i, (kind, _, _) in enumerate(self.parts):
                if kind == TABLE and t_proc[i] < fastest_table:
                    fastest_table = t_proc[i]
            for i in p_bd:
                if self.parts[i][0] == CUBE and t_proc[i] < fastest_table:
                    chosen = i
                    break
            if chosen < 0:
                # ... else the slowest TABLE partition in P_BD: the first in FOR-loop order
                for i in range(len(self.parts)):
                    if self.parts[i][0] == TABLE and i in p_bd:
                        chosen = i
                        break
            if chosen < 0:
                # P_BD holds only CUBE partitions slower than the fastest TABLE partition
                # (which misses the deadline): the earliest response among P_BD (R22)
                chosen = min(p_bd, key=lambda i: (t_r[i], i))
        else:
            # 6.) nothing meets the deadline: min |T_D - T_R| = the earliest response (R23)
            best = INF
            for i in range(len(self.parts)):
                if t_r[i] < best:
                    best = t_r[i]
                    chosen = i
        if chosen < 0:
            return (-1, 0, INF, t_d, INF)
        translated = 1 if (self.parts[chosen][1] and t_trans > 0) else 0
        if translated:
            self.t_q_trans = self.t_q_trans + t_trans
        # queue update: the partition is busy until this query's response time (R20)
        self.t_q[chosen] = t_r[chosen]
        return (chosen, translated, t_r[chosen], t_d, t_proc[chosen])

    def complete(self, partition, t_est, t_real):
        """the real processing time is compared with the estimate and
        the difference updates T_Q of the queue that processed the query."""
        self.t_q[partition] = self.t_q[partition] + (t_real - t_est)
