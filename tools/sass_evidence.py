#!/usr/bin/env python3
"""SASS evidence for the round's build: per kernel, counts of the instructions the design relies on
(bulk copies UBLKCP, mbarrier SYNCS.*, LDG.256 / LDS.128 vector loads, shuffles, fp64 adds, ...)
and the first lines that use them.  usage: sass_evidence.py > profiles/sass/sass_r02_memory_ops.txt"""
import collections
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_ipps_malikrse12_b200", "libolap_b200.so")
KERNELS = [  # (label, mangled-name regex)
    ("tile_reduce_kernel<float, AccF>", r"tile_reduce_kernelIfNS_4AccF"),
    ("tile_reduce_kernel<int, AccI>", r"tile_reduce_kernelIiNS_4AccI"),
    ("brick_reduce_kernel<float, AccF, 1> (2x4x4 bricks)", r"brick_reduce_kernelIfNS_4AccFELi1E"),
    ("reduce_kernel<float, AccF> (item path)", r"13reduce_kernelIfNS_4AccF"),
    ("table_scan_kernel", r"table_scan_kernel"),
    ("translate_kernel", r"translate_kernel"),
]
KEEP = re.compile(r"^(UBLKCP|SYNCS|LDG|LDS|STS|STG|ATOM|RED|SHFL|REDUX|CREDUX|DADD|F2F|FADD|FMNMX|VIMNMX|PRMT|"
                  r"LOP3|IMAD|ISETP|MUFU|I2F)")


def main():
    tmp = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", LIB], cwd=tmp, capture_output=True, check=True)
    funcs = {}
    for f in sorted(os.listdir(tmp)):
        if not f.endswith(".cubin"):
            continue
        out = subprocess.run(["nvdisasm", "-c", os.path.join(tmp, f)], capture_output=True, text=True).stdout
        cur = None
        for ln in out.splitlines():
            m = re.search(r"\.section\s+\.text\.([^,\s]+)", ln)
            if m:
                cur = m.group(1)
                funcs.setdefault(cur, [])
                continue
            m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", ln)
            if m and cur:
                funcs[cur].append((m.group(1), m.group(2).strip()))
    print("# SASS evidence (cuobjdump -xelf + nvdisasm of paper_conf_ipps_malikrse12_b200/libolap_b200.so, sm_100a),")
    print("# written by tools/sass_evidence.py for the build it ran on; per kernel: instruction counts of the ops the")
    print("# design relies on (static, not executed), then the first line of each memory / barrier mnemonic")
    for label, pat in KERNELS:
        names = [n for n in funcs if re.search(pat, n)]
        if not names:
            print(f"\n== {label}: not found")
            continue
        name = names[0]
        cnt = collections.Counter()
        first = {}
        for addr, ins in funcs[name]:
            op = re.sub(r"^@!?U?P\w+\s+", "", ins).split()[0]
            if KEEP.match(op):
                cnt[op] += 1
                if op.split(".")[0] in ("UBLKCP", "SYNCS", "LDG", "LDS", "STS", "REDUX", "CREDUX") and op not in first:
                    first[op] = f"/*{addr}*/ {ins}"
        print(f"\n== {label}  ({name}, {len(funcs[name])} instructions)")
        print("   " + ", ".join(f"{k}:{v}" for k, v in sorted(cnt.items())))
        for op in sorted(first):
            print(f"   e.g. {first[op]}")


if __name__ == "__main__":
    sys.exit(main())
