#!/usr/bin/env python3
"""bench.py — OLAP sub-cube query throughput on B200 (BASELINE.json metric:
"OLAP queries/sec and achieved HBM GB/s vs 8 TB/s at 1/2/4/8 B200").

Workload (N=1): config C2a — 6-D float32 cube (16,16,16,16,16,256) = 1 GiB,
device-filled with the counter-hash generator; every step answers one batch of
4,096 synthetic queries (target fraction log-uniform in [1e-4,1], ops SUM 40% /
MIN 20% / MAX 20% / AVG 10% / COUNT 10%) with inputs resident in HBM: plan ->
persistent range-reduce -> finalize.  Each step draws a different batch.
N>1 (one rank per GPU; `--gpus N` re-launches itself under torch.distributed.run when
WORLD_SIZE is unset): every rank holds a block-cyclic dim-0 shard and the library's own
NCCL communicator (olap_comm_init_rank + olap_cube_attach_comm) exchanges the 16-B/query
partials inside olap_query_batch(_device).  Scaling (--scaling): weak (default; the global
cube (16N,16,16,16,16,256) and the global batch 4,096 N grow with N, 1 GiB and 4,096
queries' worth of cells per GPU), strong (default for C3: the 32 GiB cube and the 4,096-query
batch fixed, 32/N GiB per GPU), replica (a full cube per GPU, independent batches, no
collective: SURVEY §8(e)'s comparison point).

Prints ONE JSON line (rank 0).  `--impl reference` times the CPU oracle (the
paper's OpenMP partition analogue) on the host cores instead.
"""
from __future__ import annotations

import argparse
import functools
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

METRIC = "OLAP queries/sec and achieved HBM GB/s vs 8 TB/s at 1/2/4/8 B200"
NOMINAL_HBM_GBS = 8000.0


def env_int(k, d):
    try:
        return int(os.environ.get(k, d))
    except ValueError:
        return d


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            j = json.load(f)
        return float(j["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


DESC = {
    "C1": "4-D int32 32^4 (4 MiB, L2-resident: GB/s is L2, not HBM), 1,000 random boxes, uniform ops",
    "C2a": "6-D float32 (16,16,16,16,16,256) 1 GiB; phi log-uniform [1e-4,1], l_d=max(1,round(n_d*phi^(1/6))); "
           "ops SUM/MIN/MAX/AVG/COUNT 40/20/20/10/10",
    "C2b": "6-D float32 (16,16,32,32,32,32) 1 GiB (128-B rows: short-run stress); phi log-uniform [1e-4,1]; same ops",
    "C3": "3-D float32 (2048,2048,2048) 32 GiB; phi log-uniform [1e-5,1]; same ops",
    "C5": "3-D float32 (1024,4096,8192) 128 GiB per GPU (1 TiB at 8 GPUs); small boxes 4 KiB..4 MiB log-uniform; "
          "batches of 65,536",
}


def workload(name: str, world: int):
    cfg = synth.CONFIGS[name]
    return tuple(cfg["extents"]), cfg


def batches(name, ext, nq, count, seed0, size_extents=None):
    out = []
    for k in range(count):
        b, o = synth.config_queries(name, nq=nq, seed=seed0 + 1000 + k, extents=ext, size_extents=size_extents)
        out.append((b, o))
    return out


class Clocks:
    """nvidia-smi sampler (100 ms) started before the warm-up, so that it is emitting by the time
    the timed region starts; mark() brackets the timed region and stop() keeps the samples inside
    it (or, for a region shorter than one sample period, the samples nearest to it)."""

    FIELDS = ("timestamp,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.proc = None
        self.t0 = self.t1 = None
        self.path = os.path.join(ROOT, "gpurun_out", f"clocks_{os.getpid()}.csv")
        try:
            os.makedirs(os.path.dirname(self.path), exist_ok=True)
            self.f = open(self.path, "w")
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=self.f, stderr=subprocess.DEVNULL)
            deadline = time.time() + 5.0  # wait for the first sample (nvidia-smi start-up)
            while time.time() < deadline and os.path.getsize(self.path) == 0:
                time.sleep(0.05)
        except Exception:
            self.proc = None

    def mark(self, start: bool):
        if start:
            self.t0 = time.time()
        else:
            self.t1 = time.time()

    def stop(self):
        if self.proc is None:
            return None
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.f.close()
        import datetime as _dt
        rows = []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in open(self.path):
            parts = [p.strip() for p in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                ts = _dt.datetime.strptime(parts[0], "%Y/%m/%d %H:%M:%S.%f").timestamp()
                rows.append((ts, float(parts[1]), float(parts[2]),
                             {n for n, v in zip(names, parts[5:9]) if v.lower() in ("active", "1")}))
            except ValueError:
                continue
        if not rows:
            return None
        t0 = self.t0 if self.t0 is not None else rows[0][0]
        t1 = self.t1 if self.t1 is not None else rows[-1][0]
        inside = [r for r in rows if t0 - 0.05 <= r[0] <= t1 + 0.05]
        where = "timed region"
        if not inside:  # region shorter than the sampling period: the samples just around it
            rows.sort(key=lambda r: min(abs(r[0] - t0), abs(r[0] - t1)))
            inside = rows[:2]
            where = "nearest to the timed region"
        reasons = set().union(*[r[3] for r in inside])
        return {"sm_mhz": statistics.median([r[1] for r in inside]), "sm_max_mhz": max(r[2] for r in inside),
                "reasons": sorted(reasons), "samples": len(inside), "window": where,
                "region_s": (t1 - t0) if (self.t0 and self.t1) else None}


def _oracle_rate(run, n_total, target_s, chunk):
    """Call run(i0, i1) on consecutive chunks of a (shuffled) sample until ~target_s has passed."""
    done, t0 = 0, time.perf_counter()
    while done < n_total and (time.perf_counter() - t0) < target_s:
        n = min(chunk, n_total - done)
        run(done, done + n)
        done += n
    return done, time.perf_counter() - t0


def cpu_baseline(name, ext_global, cfg, seed, target_s=12.0, max_queries=None, single_s=4.0):
    """The oracle as it stands (-O3 -march=native, oracle/__init__.py CFLAGS), timed on the host
    cores twice, as the paper does (1 thread and all cores): OpenMP over queries
    (schedule dynamic) on every core for ~target_s, and one thread for ~single_s, each on a
    random sample of the same batch the GPU answers (deviation from SURVEY §8(d)'s whole C2 batch:
    its 4,096 queries read ~440 GiB, minutes of CPU time; the sample is uniform over the batch)."""
    import oracle
    ext = cfg["extents"]  # a one-GPU cube; the oracle evaluates the global cube semantics on it
    ncells = int(np.prod(ext))
    dt = np.dtype(cfg["dtype"])
    # materialise the cube on the host when it is small; else the oracle recomputes cells procedurally
    cells = _host_cells(tuple(ext), dt.str, cfg["seed"]) if ncells * 4 <= (2 << 30) else None
    b, o = synth.config_queries(name, nq=cfg["nq"], seed=seed, extents=ext)
    perm = np.random.default_rng(seed).permutation(len(b))
    if max_queries is not None:
        perm = perm[:max_queries]
    b, o = b[perm], o[perm]
    threads = oracle.max_threads()
    vol = np.prod(b[:, :, 1] - b[:, :, 0] + 1, axis=1)
    read = np.where(o != synth.COUNT, vol, 0)

    def run(nthreads):
        def f(i0, i1):
            if cells is not None:
                oracle.query(ext, b[i0:i1], o[i0:i1], cells, nthreads=nthreads)
            else:
                oracle.query(ext, b[i0:i1], o[i0:i1], dtype=dt, gen=oracle.GEN_UNIFORM, seed=cfg["seed"],
                             nthreads=nthreads)
        return f

    done, t_used = _oracle_rate(run(threads), len(b), target_s, max(threads, 8))
    gib = float(read[:done].sum()) * 4 / 2**30
    d1, t1 = _oracle_rate(run(1), len(b), single_s, 1) if single_s > 0 else (0, 0.0)
    gib1 = float(read[:d1].sum()) * 4 / 2**30
    return {
        "value": done / t_used, "unit": "queries/s", "cores": threads, "kind": "oracle",
        "gbs": gib * 2**30 / t_used / 1e9,
        "sample": f"{done} queries drawn uniformly from a {name} batch on the 1-GPU cube {tuple(ext)}, "
                  f"{gib:.1f} GiB read in {t_used:.1f} s, OpenMP over queries on {threads} threads"
                  + ("" if cells is not None else ", cells recomputed by the oracle's generator"),
        "single_thread": ({"value": d1 / t1, "unit": "queries/s", "cores": 1, "gbs": gib1 * 2**30 / t1 / 1e9,
                           "sample": f"{d1} queries of the same sample, {gib1:.2f} GiB in {t1:.1f} s"}
                          if d1 else None),
        "build": "g++ " + " ".join(oracle.CFLAGS),
        "host": host_info(),
    }


@functools.lru_cache(maxsize=2)
def _host_cells(ext, dtype_str, seed):
    return synth.uniform_cells(int(np.prod(ext)), np.dtype(dtype_str), seed)


def _traffic(workload, kernel="reduce_kernel"):
    """DRAM read+write bytes per launch of `kernel` on `workload` from ncu (profiles/traffic.json)."""
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        with open(tp) as f:
            v = json.load(f).get(workload)
        if isinstance(v, dict):
            return v.get(kernel)
        return v if kernel == "reduce_kernel" else None
    return None


def host_info():
    model = ""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "cpu": model, "OMP_NUM_THREADS": os.environ.get("OMP_NUM_THREADS")}


def run_reference(args, rank, world):
    if rank != 0:
        return 0
    ext, cfg = workload(args.workload, 1)
    steps, warm = args.steps, args.warmup
    # each step: a bounded sample of one batch (the full batch is ~444 GiB of reads)
    vals = []
    per_step = max(1.0, 60.0 / max(1, steps + warm))
    for k in range(warm + steps):
        cb = cpu_baseline(args.workload, ext, cfg, seed=cfg["seed"] + 1000 + k, target_s=per_step, single_s=0)
        if k >= warm:
            vals.append(cb)
    q = sum(v["value"] for v in vals) / len(vals)
    gbs = sum(v["gbs"] for v in vals) / len(vals)
    line = {
        "impl": "reference", "metric": METRIC, "value": q, "unit": "queries/s", "n_gpus": world,
        "steps": steps, "warmup": warm, "ms_per_step": 1000.0 / q * cfg["nq"], "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "i32" if cfg["dtype"] == np.int32 else "f32",
        "data": "synthetic",
        "config": {"workload": args.workload, "extents": list(ext), "batch": cfg["nq"],
                   "note": "oracle on a bounded sample per step; ms_per_step extrapolated to a full batch"},
        "gbs": gbs,
        "cpu_baseline": {"value": q, "unit": "queries/s", "cores": vals[0]["cores"], "kind": "oracle",
                         "sample": vals[0]["sample"]},
        "e2e": {"value": q, "unit": "queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def cpu_baseline_c4(ext, cols, members, ids_host, qty, queries, target_s=12.0, single_s=4.0):
    """C4's oracle leg: the oracle's std::map dictionaries turn each query's strings into ranges
    (readings R11/R13), and oracle.query answers them on the quantity cube the oracle built from
    the same fact rows (oracle.factbuild; build not timed).  All cores (OpenMP over queries) and
    one thread, on a uniform sample of the batch."""
    import oracle
    cube = oracle.factbuild(ext, ids_host, qty, np.zeros(ext, np.int32))
    od = [oracle.Dict(members[c]) for c in cols]
    threads = oracle.max_threads()
    perm = np.random.default_rng(17).permutation(len(queries))

    def ranges_of(qs):
        out = np.zeros((len(qs), len(cols), 2), np.int64)
        for qi, q in enumerate(qs):
            for di, c in enumerate(cols):
                cond = q.get(c)
                if cond is None:
                    out[qi, di] = (0, ext[di] - 1)
                elif isinstance(cond, tuple):
                    out[qi, di] = (od[di].bound(cond[0]), od[di].bound(cond[1], upper=True) - 1)
                else:
                    i = int(od[di].translate([cond])[0])
                    out[qi, di] = (i, i) if i >= 0 else (1, 0)
        return out

    def run(nthreads):
        def f(i0, i1):
            qs = [queries[j] for j in perm[i0:i1]]
            oracle.query(ext, ranges_of(qs), np.array([q["op"] for q in qs], np.int32), cube, nthreads=nthreads)
        return f

    done, t = _oracle_rate(run(threads), len(queries), target_s, max(threads, 8))
    d1, t1 = _oracle_rate(run(1), len(queries), single_s, 1)
    return {"value": done / t, "unit": "queries/s", "cores": threads, "kind": "oracle",
            "sample": f"{done} of the batch's {len(queries)} text queries (uniform sample): oracle dictionaries + "
                      f"oracle.query on the oracle-built 4.5 GiB quantity cube, {t:.1f} s, OpenMP over queries",
            "single_thread": {"value": d1 / t1, "unit": "queries/s", "cores": 1,
                              "sample": f"{d1} queries, {t1:.1f} s"} if d1 else None,
            "build": "g++ " + " ".join(oracle.CFLAGS), "host": host_info()}


def run_c4(args, rank, world):
    """C4: TPC-DS store_sales-shaped workload.  Per step, 10,000 text queries (a d_date range
    + 0-3 equality predicates on store / class / state, 5% misses, random op) are translated
    on the GPU through the four dictionaries into ranges (olap_text_ranges_device) and answered
    on the quantity cube (olap_query_batch_device).  The cubes are built on the GPU from 2^26
    synthetic fact rows (olap_cube_add_facts_device; build time reported, not timed)."""
    import torch

    import paper_conf_ipps_malikrse12_b200 as olap

    if world > 1:
        raise SystemExit("C4 is a single-GPU workload")
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    members = synth.tpcds_members()
    cols = ["ca_state", "i_class", "s_store_id", "d_date"]
    dicts = [olap.Dict(members[c]) for c in cols]
    ext = tuple(len(members[c]) for c in cols)
    nrows = 1 << 26
    facts, qty, cents = synth.tpcds_facts(nrows, members)
    # bulk encoding ("every text column is converted to integer column"): each
    # raw string column of the fact table is copied to the GPU and translated row by row through
    # its dictionary (olap_dict_translate_device) into the id matrix the cube build reads
    d_ids = torch.empty((len(cols), nrows), dtype=torch.int32, device=dev)
    enc_s, enc_bytes, enc_miss = 0.0, 0, torch.zeros(1, dtype=torch.int64, device=dev)
    for i, c in enumerate(cols):
        raw, offs = synth.text_column(members[c], facts[c])
        d_raw, d_offs = torch.from_numpy(raw).to(dev), torch.from_numpy(offs).to(dev)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        olap.translate_device([dicts[i]], None, d_raw, d_offs, nrows, d_ids[i], enc_miss)
        torch.cuda.synchronize()
        enc_s += time.perf_counter() - t0
        enc_bytes += raw.nbytes
        del d_raw, d_offs, raw, offs
    if int(enc_miss.item()):
        raise SystemExit("bulk encoding: a fact string is missing from its dictionary")
    cube = olap.Cube(ext, np.int32)
    cube.fill(olap.GEN_AFFINE, 0, np.zeros(len(ext) + 1))
    torch.cuda.synchronize()
    tb0 = time.perf_counter()
    cube.add_facts_device(d_ids, torch.from_numpy(qty).to(dev))
    torch.cuda.synchronize()
    build_s = time.perf_counter() - tb0
    # the net_paid cube (float32): the deterministic build (sort by cell, fp64 per cell, one rounding)
    paid = olap.Cube(ext, np.float32)
    paid.fill(olap.GEN_AFFINE, 0, np.zeros(len(ext) + 1))
    d_cents = torch.from_numpy(cents).to(dev)
    torch.cuda.synchronize()
    tb0 = time.perf_counter()
    paid.add_facts_device(d_ids, d_cents)
    torch.cuda.synchronize()
    build_f_s = time.perf_counter() - tb0
    ids_host = d_ids.cpu().numpy() if not args.no_cpu_baseline else None  # the oracle leg's fact rows
    del d_ids, d_cents, paid
    nq = 10_000
    steps, warm = args.steps, args.warmup
    batches_ = []
    for k in range(warm + steps):
        qs = synth.tpcds_queries(nq, members, seed=synth.SEED_BASE + 3 + 7919 * (k + 1))
        conds = [[q.get(c) if c != "d_date" else q[c] for c in cols] for q in qs]
        ops = np.array([q["op"] for q in qs], np.int32)
        kinds, first, rin, buf, offs = olap.pack_text_conditions(conds, len(cols))
        batches_.append(dict(conds=conds, ops=ops, host=(kinds, rin, buf, offs), kinds=torch.from_numpy(kinds).to(dev),
                             first=torch.from_numpy(first).to(dev), buf=torch.from_numpy(buf.copy()).to(dev),
                             offs=torch.from_numpy(offs).to(dev), nkeys=len(offs) - 1,
                             d_ops=torch.from_numpy(ops).to(dev)))
    ranges = torch.empty((nq, len(cols), 2), dtype=torch.int64, device=dev)
    res = torch.empty(nq * olap.RESULT_DTYPE.itemsize, dtype=torch.uint8, device=dev)
    miss = torch.zeros(1, dtype=torch.int64, device=dev)
    stream = torch.cuda.Stream(device=dev)

    def step(k, t_split=None):
        b = batches_[k]
        olap.text_ranges_device(dicts, ext, nq, b["kinds"], b["first"], None, b["buf"], b["offs"], b["nkeys"],
                                ranges, miss, stream=stream)
        if t_split is not None:
            t_split.record(stream)
        cube.query_device(ranges, b["d_ops"], res, nq=nq, stream=stream)

    for k in range(warm):
        step(k)
    stream.synchronize()
    cube.profile(True)
    k0 = cube.stats()[0]
    f0 = olap.lib.olap_finalize_launches()
    clocks = Clocks(0)
    clocks.mark(True)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True),
           torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for i, k in enumerate(range(warm, warm + steps)):
        ev[i][0].record(stream)
        step(k, ev[i][1])
        ev[i][2].record(stream)
    e1.record(stream)
    e1.synchronize()
    clocks.mark(False)
    elapsed = e0.elapsed_time(e1)
    clk = clocks.stop()
    trans_ms = sum(a.elapsed_time(b) for a, b, _ in ev)
    c4_kernel = "tile_reduce_kernel" if cube.tile_stats()[3] else "reduce_kernel"
    gpu_launches = cube.stats()[0] - k0 + olap.lib.olap_finalize_launches() - f0 + steps  # + one text_ranges_kernel
    reduce_ms, launches, alg_bytes = cube.profile_read()
    cube.profile(False)
    nkeys = sum(batches_[k]["nkeys"] for k in range(warm, warm + steps))
    # end to end through the host-buffer API: olap_text_ranges + olap_query_batch
    t0 = time.perf_counter()
    e2e_steps = max(1, args.e2e_steps)
    for k in range(e2e_steps):
        b = batches_[warm + (k % steps)]
        boxes, _ = olap.text_ranges_packed(dicts, ext, nq, *b["host"])   # strings already in the C-ABI layout
        cube.query(boxes, b["ops"])
    e2e_s = time.perf_counter() - t0
    peak, peak_src = measured_peaks()
    achieved = (alg_bytes / max(launches, 1)) / (reduce_ms / max(launches, 1) / 1e3) / 1e9 if reduce_ms else 0.0
    cpu = None
    if ids_host is not None:
        qs0 = synth.tpcds_queries(nq, members, seed=synth.SEED_BASE + 3 + 7919 * (warm + 1))
        cpu = cpu_baseline_c4(ext, cols, members, ids_host, qty, qs0)
    line = {
        "metric": METRIC, "value": nq * steps / (elapsed / 1e3), "unit": "queries/s", "n_gpus": 1, "steps": steps,
        "warmup": warm, "ms_per_step": elapsed / steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "i32", "data": "synthetic",
        "config": {"workload": "C4", "extents": list(ext), "dims": cols, "fact_rows": nrows, "batch": nq,
                   "queries": "d_date range + 0-3 equality predicates (store/class/state, 5% misses), random op; "
                              "text translated on the GPU each step",
                   "cube_build_s": build_s, "float_cube_build_s": build_f_s,
                   "bulk_encoding": {"rows": nrows, "columns": len(cols), "s": enc_s,
                                     "keys_per_s": nrows * len(cols) / enc_s, "string_bytes": enc_bytes,
                                     "api": "olap_dict_translate_device over the raw fact-table string columns"},
                   "l2": "no flush: 4.5 GiB cube > L2"},
        "gbs": alg_bytes / (elapsed / 1e3) / 1e9,
        "translation": {"keys_per_s": nkeys / (trans_ms / 1e3), "share_of_step": trans_ms / elapsed,
                        "paper_share": 0.07},
        "roofline": cube_roofline("C4", c4_kernel, achieved, reduce_ms / max(launches, 1) / 1e3, clk,
                                  alg_bytes / max(launches, 1), reduce_ms / elapsed if elapsed else None),
        "gpu_launches": int(gpu_launches), "clocks": clk,
        "e2e": {"value": nq * e2e_steps / e2e_s, "unit": "queries/s",
                "h2d_bytes_per_step": int(sum(x.nbytes for x in batches_[warm]["host"])) + int(nq * 4 * 2 * 16 + nq * 4),
                "d2h_bytes_per_step": int(nq * 4 * 2 * 8 + nq * 24),
                "api": "olap_text_ranges + olap_query_batch (host buffers; conditions pre-packed in the C-ABI layout)"},
        "cpu_baseline": cpu,
    }
    print(json.dumps(line), flush=True)
    return 0


def cpu_baseline_table(columns, queries, target_s=12.0, single_s=4.0):
    """T's oracle leg: oracle.tablescan (the plain row loop of Q_D, Eq. 11-12) over the same 2^26
    host columns, OpenMP over queries on all cores and one thread, on a uniform batch sample."""
    import oracle
    threads = oracle.max_threads()
    perm = np.random.default_rng(19).permutation(len(queries))

    def run(nthreads):
        def f(i0, i1):
            oracle.tablescan(columns, [queries[j] for j in perm[i0:i1]], nthreads=nthreads)
        return f

    done, t = _oracle_rate(run(threads), len(queries), target_s, max(threads, 8))
    d1, t1 = _oracle_rate(run(1), len(queries), single_s, 1)
    return {"value": done / t, "unit": "queries/s", "cores": threads, "kind": "oracle",
            "sample": f"{done} of the batch's {len(queries)} queries (uniform sample), oracle.tablescan over the "
                      f"2^26-row host columns, {t:.1f} s, OpenMP over queries",
            "single_thread": {"value": d1 / t1, "unit": "queries/s", "cores": 1,
                              "sample": f"{d1} queries, {t1:.1f} s"} if d1 else None,
            "build": "g++ " + " ".join(oracle.CFLAGS), "host": host_info()}


def run_table(args, rank, world):
    """T: the paper's own GPU path — queries Q_D (Eq. 11) over a column-store
    fact table of 2^26 store_sales-shaped rows (4 dimension-id columns + quantity int32 +
    net_paid float32).  Per step one batch of 4,096 queries (d_date range + 0-3 equality
    predicates on store / class / state, random op on quantity or net_paid), answered by
    one shared scan (olap_table_query_batch_device)."""
    import torch

    import paper_conf_ipps_malikrse12_b200 as olap

    if world > 1:
        raise SystemExit("T is a single-GPU workload")
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    members = synth.tpcds_members()
    cols = ["ca_state", "i_class", "s_store_id", "d_date"]
    card = [len(members[c]) for c in cols]
    nrows = 1 << 26
    facts, qty, cents = synth.tpcds_facts(nrows, members)
    table = olap.Table(nrows, [np.int32] * 4 + [np.int32, np.float32])
    # ids must be dictionary ranks: translate members through the GPU dictionaries once (bulk encoding)
    dicts = [olap.Dict(members[c]) for c in cols]
    host_cols = []
    for i, c in enumerate(cols):
        rank = dicts[i].translate(members[c])[0]
        host_cols.append(rank[facts[c]].astype(np.int32))
        table.load_column(i, host_cols[-1])
    table.load_column(4, qty)
    table.load_column(5, cents)
    host_cols += [qty, cents]
    nq = 4096
    steps, warm = args.steps, args.warmup
    rng = np.random.default_rng(synth.SEED_BASE + 9)
    host, devb = [], []
    evals = []
    for k in range(warm + steps):
        qs = []
        for _ in range(nq):
            a, b = sorted(rng.integers(0, card[3], size=2))
            conds = [(3, int(a), int(b))]
            for ci in range(3):
                if rng.random() < 0.5:
                    v = int(rng.integers(0, card[ci]))
                    conds.append((ci, v, v))
            qs.append((conds, int(rng.integers(4, 6)), int(rng.integers(0, 5))))
        host.append(qs)
        off, ca, dcol, ops = olap.pack_table_queries(qs)
        devb.append(tuple(torch.from_numpy(x.view(np.uint8) if x.dtype.names else x).to(dev)
                          for x in (off, ca, dcol, ops)))
        evals.append(sum(len(q[0]) + 1 for q in qs))
    res = torch.empty(nq * olap.RESULT_DTYPE.itemsize, dtype=torch.uint8, device=dev)
    stream = torch.cuda.Stream(device=dev)
    for k in range(warm):
        table.query_device(nq, *devb[k], res, stream=stream)
    stream.synchronize()
    table.profile(True)
    clocks = Clocks(0)
    clocks.mark(True)
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for k in range(warm, warm + steps):
        table.query_device(nq, *devb[k], res, stream=stream)
    e1.record(stream)
    e1.synchronize()
    clocks.mark(False)
    elapsed = e0.elapsed_time(e1)
    scan_ms, scan_n = table.profile_read()
    table.profile(False)
    clk = clocks.stop()
    # Eq. 12 cost model of the paper's design: each query reads its C_QD columns whole
    paper_bytes = sum(evals[warm:]) * nrows * 4
    col_evals = sum(evals[warm:]) * nrows  # (query, row, column) evaluations
    # issue-rate bound: 148 SMs x 4 schedulers x 32 lanes x 1.965 GHz = 37.2e12 lane-instr/s, >= 3 per evaluation
    peak_evals = 148 * 4 * 32 * 1.965e9 / 3
    t0 = time.perf_counter()
    e2e_steps = max(1, args.e2e_steps)
    for k in range(e2e_steps):
        table.query(host[warm + (k % steps)])
    e2e_s = time.perf_counter() - t0
    achieved = col_evals / (elapsed / 1e3)
    cpu = None
    if not args.no_cpu_baseline:
        cpu = cpu_baseline_table(host_cols, host[warm])
    # the columns the batch references, each read from HBM once per batch by the shared scan
    used_cols = sorted({c for q in host[warm] for c in [x[0] for x in q[0]] + [q[1]]})
    col_bytes = len(used_cols) * nrows * 4
    peak, peak_src = measured_peaks()
    line = {
        "metric": METRIC, "value": nq * steps / (elapsed / 1e3), "unit": "queries/s", "n_gpus": 1, "steps": steps,
        "warmup": warm, "ms_per_step": elapsed / steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "i32+f32", "data": "synthetic",
        "config": {"workload": "T", "fact_rows": nrows, "columns": cols + ["ss_quantity", "ss_net_paid"],
                   "batch": nq, "queries": "d_date range + 0-3 equality predicates, op on quantity or net_paid",
                   "l2": "columns (1.6 GB) > L2; staged once per batch"},
        "paper_eq12_gbs": paper_bytes / (elapsed / 1e3) / 1e9,
        "roofline": dict(issue_roofline("T", "table_scan_kernel", scan_ms / max(scan_n, 1) / 1e3,
                                        (clk or {}).get("sm_mhz") or 1965.0),
                         traffic=_traffic("T", "table_scan_kernel"),
                         scan_share_of_step=scan_ms / elapsed if elapsed else None,
                         note="the shared scan reads every referenced column once per batch (hbm below) and then "
                              "evaluates every (query, row) from shared memory: instruction issue binds it (ncu); "
                              "kernel time from CUDA events around table_scan_kernel (olap_table_profile)",
                         hbm={"achieved": col_bytes / (elapsed / steps / 1e3) / 1e9, "peak": peak, "unit": "GB/s",
                              "frac": col_bytes / (elapsed / steps / 1e3) / 1e9 / peak, "peak_source": peak_src,
                              "note": "algorithmic bytes = the referenced columns, read once per batch"}),
        "effective_evals": {"value": achieved, "unit": "(query,row,column) evaluations/s (Eq. 12, dense)",
                            "frac_of_issue_bound": achieved / peak_evals,
                            "issue_bound": "148 SMs x 4 x 32 lanes x 1.965 GHz / 3 instr per evaluation; the "
                                           "sparse per-row checks skip most evaluations, so this is an "
                                           "effective rate, not hardware utilisation (can exceed 1)"},
        "gpu_launches": int(steps * 4), "clocks": clk,  # prep, order, scan, final per step
        "e2e": {"value": nq * e2e_steps / e2e_s, "unit": "queries/s", "api": "olap_table_query_batch (host buffers)"},
        "cpu_baseline": cpu,
    }
    print(json.dumps(line), flush=True)
    return 0


def run_resolution(args, rank, world):
    """R: the multi-resolution cube set (Eq. 2).  The C4
    quantity cube at day resolution (52,100,128,1826) is rolled up on the GPU to month (60)
    and year (5) resolution.  Each step is a batch of 10,000 queries whose date condition is
    given in years, months or days (1/3 each) with 0-3 equality predicates; olap_cubeset_query
    answers each from the cube of its resolution R = max r_i (Eq. 2).  The same batch answered
    entirely on the day cube is reported beside it (`day_cube_only`)."""
    import torch

    import paper_conf_ipps_malikrse12_b200 as olap

    if world > 1:
        raise SystemExit("R is a single-GPU workload")
    torch.cuda.set_device(0)
    members = synth.tpcds_members()
    cols = ["ca_state", "i_class", "s_store_id", "d_date"]
    card = [len(members[c]) for c in cols]
    ident = lambda n: np.arange(n, dtype=np.int32)
    levels = [[ident(card[i])] * 3 for i in range(3)] + [synth.date_hierarchy()]
    h = olap.Hierarchy(levels)
    nrows = 1 << 26
    facts, qty, _ = synth.tpcds_facts(nrows, members)
    dicts = [olap.Dict(members[c]) for c in cols]
    ids = np.stack([dicts[i].translate(members[c])[0][facts[c]] for i, c in enumerate(cols)]).astype(np.int32)
    day = olap.Cube(h.extents(2), np.int32)
    day.fill(olap.GEN_AFFINE, 0, np.zeros(5))
    day.add_facts_device(torch.from_numpy(ids).cuda(), torch.from_numpy(qty).cuda())
    torch.cuda.synchronize()
    cubes = {2: day}
    tb = time.perf_counter()
    for lvl in (1, 0):
        cubes[lvl] = olap.Cube(h.extents(lvl), np.int32)
        h.rollup(day, 2, cubes[lvl], lvl, olap.SUM)
    rollup_s = time.perf_counter() - tb
    cs = olap.CubeSet(h)
    for lvl, c in cubes.items():
        cs.add(lvl, c)
    nq = 10_000
    rng = np.random.default_rng(synth.SEED_BASE + 11)
    steps, warm = args.steps, args.warmup
    batches_ = []
    for _ in range(warm + steps):
        lv = np.zeros((nq, 4), np.int32)
        rr = np.zeros((nq, 4, 2), np.int64)
        ops = rng.choice(np.array([olap.SUM, olap.MIN, olap.MAX, olap.AVG, olap.COUNT], np.int32), size=nq)
        for q in range(nq):
            r = int(rng.integers(0, 3))
            n = len(np.unique(levels[3][r]))
            lv[q, :] = 0
            lv[q, 3] = r
            rr[q, 3] = sorted(rng.integers(0, n, size=2))
            for d in range(3):
                if rng.random() < 0.5:
                    v = int(rng.integers(0, card[d]))
                    rr[q, d] = (v, v)
                else:
                    rr[q, d] = (0, card[d] - 1)
        batches_.append((rr, lv, ops))
    for k in range(warm):
        cs.query(*batches_[k])
    torch.cuda.synchronize()
    k0 = sum(c.stats()[0] for c in cubes.values())
    t0 = time.perf_counter()
    used_hist = np.zeros(3, np.int64)
    for k in range(warm, warm + steps):
        _, used = cs.query(*batches_[k])
        used_hist += np.bincount(used[used >= 0], minlength=3)
    routed_s = time.perf_counter() - t0
    launches = sum(c.stats()[0] for c in cubes.values()) - k0
    # this line is host-bound (routing, many small synchronous batches) and a running nvidia-smi
    # sampler slows such a loop ~2.6x (driver contention, measured): the clocks come from a second,
    # identical pass over the same batches with the sampler on
    clocks = Clocks(0)
    clocks.mark(True)
    t0 = time.perf_counter()
    for k in range(warm, warm + steps):
        cs.query(*batches_[k])
    sampled_s = time.perf_counter() - t0
    clocks.mark(False)
    clk = clocks.stop()
    if clk is not None:
        clk["pass"] = f"repeat of the timed loop with the sampler running ({nq * steps / sampled_s:.0f} q/s there)"
    # the same queries answered on the day cube only (conditions converted to days)
    conv = [(h.convert(b[0], b[1], 2), b[2]) for b in batches_]
    for k in range(warm):
        day.query(*conv[k])
    t0 = time.perf_counter()
    for k in range(warm, warm + steps):
        day.query(*conv[k])
    day_s = time.perf_counter() - t0
    line = {
        "metric": METRIC, "value": nq * steps / routed_s, "unit": "queries/s", "n_gpus": 1, "steps": steps,
        "warmup": warm, "ms_per_step": routed_s / steps * 1e3, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "i32", "data": "synthetic",
        "config": {"workload": "R", "levels": {"year": h.extents(0), "month": h.extents(1), "day": h.extents(2)},
                   "batch": nq, "queries": "date condition in years / months / days (1/3 each) + 0-3 equality "
                   "predicates, random op; host-buffer API timed end to end",
                   "rollup_s": rollup_s, "queries_per_level_used": used_hist.tolist()},
        "day_cube_only": {"value": nq * steps / day_s, "unit": "queries/s"},
        "e2e": {"value": nq * steps / routed_s, "unit": "queries/s", "api": "olap_cubeset_query (host buffers)"},
        "cpu_baseline": None, "roofline": None, "gpu_launches": int(launches), "clocks": clk,
        "note": "NEXT #3 (cube set + Eq. 2 routing): host-timed through the public API (routing is host logic, "
                "every routed sub-batch an olap_query_batch); no roofline (the per-cube kernels are the C1/C2 "
                "paths) and no CPU baseline for this secondary line",
    }
    print(json.dumps(line), flush=True)
    return 0




def smem_peak_gbs(sm_mhz):
    """Shared-memory read bandwidth of one B200 at `sm_mhz`: the bytes per SM clock MEASURED by
    tools/smem_peak.cu (profiles/smem_peak.json) x 148 SMs; 128 B/clk/SM if that file is missing."""
    p = os.path.join(ROOT, "profiles", "smem_peak.json")
    bpc, src = 128.0, "derived: 32 banks x 4 B per clock per SM (no measurement found)"
    if os.path.exists(p):
        with open(p) as f:
            j = json.load(f)
        bpc = float(j["bytes_per_clk_per_sm"])
        src = f"measured: {bpc:.1f} B/clk/SM ({j['how']}) x 148 SMs x {sm_mhz:.0f} MHz (median SM clock, timed region)"
    return bpc * 148 * sm_mhz * 1e6 / 1e9, src


def issue_roofline(workload, kernel, kern_s, sm_mhz):
    """Instruction-issue roofline of an issue-bound kernel: warp instructions per launch (ncu, the same
    bench batch, profiles/traffic.json '<kernel>:inst') / the launch's CUDA-event time, against
    148 SMs x 4 SM sub-partitions x 1 warp instruction per clock at the measured SM clock."""
    inst = _traffic(workload, kernel + ":inst")
    peak = 148 * 4 * sm_mhz * 1e6
    ach = inst / kern_s if (inst and kern_s) else None
    return {"bound": "issue", "achieved": ach, "peak": peak, "unit": "warp-instr/s",
            "frac": (ach / peak) if ach else None, "kernel": kernel,
            "inst_per_launch": inst,
            "peak_source": f"derived: 148 SMs x 4 schedulers x 1 warp instruction/clk x {sm_mhz:.0f} MHz (median SM "
                           "clock of the timed region; B200_PROFILING.md / Blackwell guide: one issue per SMSP per "
                           "clock)"}


def cube_roofline(workload, kernel, achieved, kern_s, clk, alg_bytes_launch, share, with_traffic=True):
    """The roofline object of a cube workload's dominant kernel (achieved = algorithmic bytes, Eq. 3,
    of one launch / that launch's CUDA-event time).  tile_reduce_kernel serves every query from
    shared memory: bound smem (measured peak); brick_reduce_kernel streams 128-B bricks from HBM:
    bound hbm; the item path is HBM / L2 (C1: L2-resident by design)."""
    hbm_peak, hbm_src = measured_peaks()
    traffic = _traffic(workload, kernel) if with_traffic else None
    dram = {"gbs": traffic / kern_s / 1e9, "frac_of_hbm": traffic / kern_s / 1e9 / hbm_peak,
            "source": "ncu dram__bytes_read.sum + dram__bytes_write.sum per launch (profiles/traffic.json) / the "
                      "kernel's CUDA-event time here"} if (traffic and kern_s) else None
    sm_mhz = (clk or {}).get("sm_mhz") or 1965.0
    if kernel == "tile_reduce_kernel":
        r = issue_roofline(workload, kernel, kern_s, sm_mhz)
        speak, ssrc = smem_peak_gbs(sm_mhz)
        r["note"] = ("tile-shared scan: each 48-KiB cube tile is staged into shared memory once per batch "
                     "(cp.async.bulk) with its slot trees; every query reduces its cells of the tile from there (run "
                     "interiors as O(log) tree entries, edge cells one by one), so neither HBM nor shared-memory "
                     "bandwidth binds it: ncu shows instruction issue as the limit (profiles/).  achieved = the "
                     "launch's warp instructions (ncu smsp__inst_executed.sum of the same batch, profiles/"
                     "traffic.json) / its CUDA-event time here; peak = 148 SMs x 4 schedulers x 1 warp-instr/clk")
        r["eq3"] = {"achieved": achieved, "unit": "GB/s",
                    "note": "the paper's cost model (Eq. 3: V_q*4 bytes per non-COUNT query) per second of the kernel",
                    "smem": {"peak": speak, "frac": achieved / speak, "peak_source": ssrc},
                    "hbm": {"peak": hbm_peak, "frac": achieved / hbm_peak, "peak_source": hbm_src}}
        r["traffic"] = traffic
    elif kernel == "brick_reduce_kernel":
        r = {"bound": "hbm", "achieved": achieved, "peak": hbm_peak, "unit": "GB/s", "frac": achieved / hbm_peak,
             "traffic": traffic, "kernel": kernel, "peak_source": hbm_src,
             "note": "bricked layout: achieved = algorithmic bytes (V_q*4, Eq. 3) / brick_reduce_kernel time; the "
                     "kernel reads whole 128-B bricks (one DRAM fetch line each), so traffic exceeds the algorithmic "
                     "bytes by the edge bricks' unselected cells (dram.gbs is what the HBM actually moved)"}
    else:
        r = {"bound": "hbm" if workload != "C1" else "l2", "achieved": achieved, "peak": hbm_peak, "unit": "GB/s",
             "frac": achieved / hbm_peak, "traffic": traffic, "kernel": kernel, "peak_source": hbm_src,
             "note": "item path: achieved = algorithmic bytes (V_q*4, Eq. 3) / reduce-kernel time; frac > 1 is L2 "
                     "reuse (items run in cube-address order)" +
                     ("; C1's 4 MiB cube is L2-resident by design: the HBM peak is only a reference"
                      if workload == "C1" else "")}
    r.update({"dram": dram, "algorithmic_bytes_per_launch": alg_bytes_launch, "reduce_share_of_step": share})
    return r


def default_scaling(name):
    # C3 (32 GiB) fits one B200: the fixed global cube is split N ways (strong); the other cube
    # workloads grow the global cube and the global batch with N (weak: fixed work per GPU)
    return "strong" if name == "C3" else "weak"


def scaled_workload(name, world, scaling):
    """(global extents, global batch) of `name` at `world` GPUs under `scaling`."""
    cfg = synth.CONFIGS[name]
    ext, nq = list(cfg["extents"]), cfg["nq"]
    if scaling == "weak" and world > 1:
        ext[0] *= world
        nq *= world
    return tuple(ext), nq


def launch_ranks(n):
    """`python bench.py --gpus N` outside torchrun: re-run this command as N ranks (one per GPU)."""
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def run_cube(args, rank, world, local):
    """C1 / C2a / C2b / C3 / C5: batches of sub-cube queries (the north_star hot path)."""
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_malikrse12_b200 as olap

    scaling = args.scaling or default_scaling(args.workload)
    if world == 1:
        scaling = "weak"  # one GPU: the config as BASELINE names it
    backend = os.environ.get("OLAP_DIST_BACKEND", "nccl")  # gloo: dry-run N ranks on one GPU
    local = local % max(torch.cuda.device_count(), 1) if backend != "nccl" else local
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    cfg = synth.CONFIGS[args.workload]
    # OLAP_BENCH_SHARDED=1 runs the N > 1 code path (a shard with the library's communicator
    # attached) at N = 1 as well: a 1-rank NCCL communicator, for testing on one GPU
    sharded = (world > 1 and scaling != "replica") or os.environ.get("OLAP_BENCH_SHARDED") == "1"
    # OLAP_BENCH_VIRTUAL_WORLD=V (one GPU, development aid): rank 0's shard of the V-GPU job -- the
    # V-fold workload, this GPU holding shard 0 of V with a 1-rank communicator -- so the per-GPU step
    # of an N-GPU run can be timed on one GPU (the line says "virtual_world"; it is not an N-GPU result)
    vworld = int(os.environ.get("OLAP_BENCH_VIRTUAL_WORLD", "0") or 0) if world == 1 else 0
    if vworld > 1:
        sharded = True
        scaling = args.scaling or default_scaling(args.workload)
    sworld = vworld if vworld > 1 else world  # the world the workload and the shard are sized for
    ext, nq = scaled_workload(args.workload, sworld, scaling if sharded else "strong")
    if args.batch:
        nq = args.batch * (sworld if (sharded and scaling == "weak") else 1)
    dtype = cfg["dtype"]
    nd = len(ext)
    layout = args.layout if args.layout != "auto" else ("brick3" if args.workload == "C5" else "row")
    lay = {"brick": olap.LAYOUT_BRICK, "brick3": olap.LAYOUT_BRICK3}.get(layout, olap.LAYOUT_ROWMAJOR)
    bricked = layout in ("brick", "brick3")
    comm = None
    if sharded:
        # this rank's block-cyclic dim-0 shard; the library's NCCL communicator does the exchange
        from paper_conf_ipps_malikrse12_b200.dist import init_comm
        vshard = int(os.environ.get("OLAP_BENCH_VIRTUAL_SHARD", "0") or 0) if vworld > 1 else rank
        cube = olap.Cube(ext, dtype, shard=(sworld, vshard, args.shard_block), device=local, layout=lay)
        if vworld <= 1:
            comm = init_comm(rank, world, local) if world > 1 else olap.Comm(olap.comm_unique_id(), 1, 0, local)
            cube.attach_comm(comm)
    else:
        cube = olap.Cube(ext, dtype, device=local, layout=lay)
    cube.fill(olap.GEN_UNIFORM, cfg["seed"])
    # replicas answer different batches; shards answer the same global batch
    seed0 = cfg["seed"] + (7919 * rank if (world > 1 and not sharded) else 0)
    # weak scaling over N GPUs: the global cube and batch grow N-fold, every query keeps the box sizes
    # of the one-GPU recipe (offsets over the global cube) -- fixed bytes and pairs per GPU per step
    weak_sizes = cfg["extents"] if (sharded and scaling == "weak" and sworld > 1) else None
    host_batches = batches(args.workload, ext, nq, args.warmup + args.steps, seed0, size_extents=weak_sizes)
    d_batches = [(torch.from_numpy(b).to(dev), torch.from_numpy(o).to(dev)) for b, o in host_batches]
    res = torch.empty(nq * olap.RESULT_DTYPE.itemsize, dtype=torch.uint8, device=dev)
    stream = torch.cuda.Stream(device=dev)

    if vworld > 1:  # shard 0's partials + finalize: the per-GPU compute of the V-GPU job, no exchange
        v_sum = torch.empty(nq, dtype=torch.int64, device=dev)
        v_ext = torch.empty(2 * nq, dtype=torch.int32, device=dev)

    def step(k):
        dr, do = d_batches[k]
        if vworld > 1:
            cube.partials_device(dr, do, v_sum, v_ext, nq=nq, stream=stream)
            olap.finalize_device(ext, dtype, nq, dr, do, v_sum, v_ext, res, stream=stream)
            return
        cube.query_device(dr, do, res, nq=nq, stream=stream)

    for k in range(args.warmup):
        step(k)
    stream.synchronize()
    graphs = None
    if args.graph and world == 1:
        # one CUDA graph per batch (plan, order, reduce, finalize), captured after the warm-up sized the workspace
        graphs = []
        gk0, gf0 = cube.stats()[0], olap.lib.olap_finalize_launches()
        for k in range(args.warmup + args.steps):
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=stream):
                cube.query_device(d_batches[k][0], d_batches[k][1], res, nq=nq, stream=torch.cuda.current_stream())
            graphs.append(g)
        torch.cuda.synchronize()
        graph_kernels = (cube.stats()[0] - gk0 + olap.lib.olap_finalize_launches() - gf0) / len(graphs)

        def step(k):  # noqa: F811
            with torch.cuda.stream(stream):
                graphs[k].replay()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    cube.profile(True)
    k0, l2_order = cube.stats()
    f0 = olap.lib.olap_finalize_launches()
    clocks = Clocks(local)
    clocks.mark(True)
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for k in range(args.warmup, args.warmup + args.steps):
        step(k)
    e1.record(stream)
    e1.synchronize()
    torch.cuda.synchronize()
    clocks.mark(False)
    elapsed_ms = e0.elapsed_time(e1)
    clk = clocks.stop()
    tiles_enabled, tile_cells, _nt, tiles_used = cube.tile_stats()
    gpu_launches = cube.stats()[0] - k0 + olap.lib.olap_finalize_launches() - f0
    if graphs is not None:
        gpu_launches = graph_kernels * args.steps
    reduce_ms, launches, alg_bytes = cube.profile_read()
    cube.profile(False)
    t = torch.tensor([elapsed_ms], dtype=torch.float64, device=dev)
    tb = torch.tensor([alg_bytes], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dist.all_reduce(tb, op=dist.ReduceOp.SUM)
    elapsed_ms = float(t.item())
    total_bytes = float(tb.item())
    total_q = nq * args.steps * (world if not sharded else 1)
    qps = total_q / (elapsed_ms / 1e3)
    gbs_total = total_bytes / (elapsed_ms / 1e3) / 1e9
    hbm_peak, hbm_src = measured_peaks()
    kern_s = reduce_ms / max(launches, 1) / 1e3
    achieved = (alg_bytes / max(launches, 1)) / kern_s / 1e9 if reduce_ms else 0.0

    # end to end through the public host-buffer C-ABI (H2D of ranges/ops, D2H of results inside):
    # olap_query_batch on every rank (on a shard with a communicator it is the library's collective)
    e2e = None
    if args.e2e_steps > 0:
        outs = np.zeros(nq, dtype=olap.RESULT_DTYPE)
        b0, o0 = host_batches[0]
        cube.query(b0, o0, out=outs)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for k in range(args.e2e_steps):
            b, o = host_batches[args.warmup + (k % args.steps)]
            cube.query(b, o, out=outs)
        e2e_t = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
        e2e_q = nq * args.e2e_steps * (world if not sharded else 1)
        e2e = {"value": e2e_q / float(e2e_t.item()), "unit": "queries/s",
               "h2d_bytes_per_step": int(nq * nd * 16 + nq * 4), "d2h_bytes_per_step": int(nq * 24),
               "api": ("olap_query_batch on this rank's shard with the library's NCCL communicator attached "
                       "(pinned H2D, shard partials, ncclAllReduce of 16 B/query, finalize, D2H; max over ranks)"
                       if sharded else "olap_query_batch (host buffers; pinned staging inside the library)")}
        if args.stream_batch:
            # the same queries as one stream through olap_query_stream (pipelined batches)
            allb = np.concatenate([host_batches[args.warmup + (k % args.steps)][0] for k in range(args.e2e_steps)])
            allo = np.concatenate([host_batches[args.warmup + (k % args.steps)][1] for k in range(args.e2e_steps)])
            cube.query_stream(allb[:nq], allo[:nq], batch=args.stream_batch)
            if world > 1:
                dist.barrier()
            t0 = time.perf_counter()
            cube.query_stream(allb, allo, batch=args.stream_batch)
            st_t = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
            if world > 1:
                dist.all_reduce(st_t, op=dist.ReduceOp.MAX)
            e2e["stream"] = {"value": len(allo) * (world if not sharded else 1) / float(st_t.item()),
                             "unit": "queries/s", "batch": args.stream_batch,
                             "api": "olap_query_stream (batch k+1 reduces while batch k exchanges / finalizes)"}

    kernel = "tile_reduce_kernel" if tiles_used else ("brick_reduce_kernel" if bricked else "reduce_kernel")
    roofline = cube_roofline(args.workload, kernel, achieved, kern_s, clk, alg_bytes / max(launches, 1),
                             reduce_ms / elapsed_ms if elapsed_ms else None, with_traffic=world == 1 and vworld <= 1)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(args.workload, ext, cfg, seed=cfg["seed"] + 1000 + args.warmup)
    if rank == 0:
        par = "1gpu" if world == 1 else (f"shard{world}" if sharded else f"replica{world}")
        line = {
            "metric": METRIC, "value": qps, "unit": "queries/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": elapsed_ms / args.steps, "higher_is_better": True,
            "scaling": "strong" if (sharded and scaling == "strong") else "weak",
            "vs_baseline": None, "dtype": "i32" if dtype == np.int32 else "f32",
            "data": "synthetic",
            "config": {"workload": args.workload, "extents": list(ext), "cube_gib_per_gpu":
                       cube.info()[1] * 4 / 2**30, "batch": nq,
                       "queries": DESC[args.workload],
                       "l2": ("no flush: C1's 4 MiB cube is L2-resident by design (flagged)" if args.workload == "C1"
                              else "no flush: cube > L2 (126 MB) and every step reads >> L2"),
                       "accumulation": ("int32 cells, int64 SUM" if dtype == np.int32 else
                                        ("f32 cells, SUM in fp32 trees (slot trees of up to 256 cells, quads of them; depth <= 10) then f64 (reading R8')"
                                         if tiles_used else
                                         ("f32 cells, SUM in fp32 trees of 8 cells of a brick then f64"
                                          if bricked else "f32 cells, f64 SUM"))),
                       "path": "tile-shared scan" if tiles_used else ("brick" if bricked else "item path"),
                       "layout": {"brick": "bricked: last two dims in 4x8-cell (128-B) bricks",
                                  "brick3": "bricked: last three dims in 2x4x4-cell (128-B) bricks (dim 0: local "
                                            "row pairs)"}.get(layout, "row-major"),
                       "parallelism": par if vworld <= 1 else f"virtual shard {vshard} of {vworld} (one GPU)",
                       "shard_block": args.shard_block if sharded else None,
                       "virtual_world": vworld if vworld > 1 else None,
                       "box_sizes": ("one-GPU recipe (weak scaling: every query reads what it reads at N = 1, "
                                     "offsets over the global cube)" if weak_sizes is not None else "config recipe"),
                       "exchange": ("none (virtual shard: partials + finalize of shard 0 only)" if vworld > 1 else
                                    ("library NCCL: ncclAllReduce of the 16-B/query partials per batch "
                                     "(olap_cube_attach_comm)" if sharded else None))},
            "gbs": gbs_total, "frac_of_nominal_8tbs": gbs_total / world / NOMINAL_HBM_GBS,
            "roofline": roofline,
            "gpu_launches": int(gpu_launches), "l2_order": l2_order,
            "clocks": clk,
            "e2e": e2e,
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        cube.close()
        if comm is not None:
            comm.close()
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=None,
                    help="GPUs (one rank each); without torchrun, N > 1 re-launches itself under torch.distributed.run")
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="C2a", choices=["C2a", "C2b", "C3", "C1", "C4", "C5", "T", "R"])
    ap.add_argument("--scaling", default=None, choices=["weak", "strong", "replica"],
                    help="N > 1: weak (global cube and batch grow with N; default), strong (fixed global cube "
                         "and batch; default for C3), replica (a full cube per GPU, independent batches)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--stream-batch", type=int, default=0,
                    help="also time the e2e queries as one olap_query_stream in batches of this size")
    ap.add_argument("--graph", action="store_true", help="replay each step as a captured CUDA graph (N=1)")
    ap.add_argument("--batch", type=int, default=0, help="queries per batch per GPU (default: the config's)")
    ap.add_argument("--shard-block", type=int, default=None,
                    help="block-cyclic dim-0 shard block b (rows; DESIGN.md §5, §8): row r lives on GPU (r / b) mod N; "
                         "default 4 for C5 (small boxes: fewer (query, GPU) splits), else 1")
    ap.add_argument("--layout", default="auto", choices=["auto", "row", "brick", "brick3"],
                    help="cube layout in HBM (auto: 2x4x4 bricks for C5's small boxes, row-major otherwise; "
                         "DESIGN.md §5)")
    args = ap.parse_args()

    rank, world, local = env_int("RANK", 0), env_int("WORLD_SIZE", 1), env_int("LOCAL_RANK", 0)
    launched = "WORLD_SIZE" in os.environ
    if args.gpus is None:
        args.gpus = world
    if args.shard_block is None:
        args.shard_block = 4 if args.workload == "C5" else 1
    if not launched and args.gpus > 1:
        return launch_ranks(args.gpus)
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}: launch one rank per GPU")
    if args.impl == "reference":
        return run_reference(args, rank, world)
    if args.workload == "C4":
        return run_c4(args, rank, world)
    if args.workload == "T":
        return run_table(args, rank, world)
    if args.workload == "R":
        return run_resolution(args, rank, world)
    return run_cube(args, rank, world, local)


if __name__ == "__main__":
    sys.exit(main())
