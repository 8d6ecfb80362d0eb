#!/usr/bin/env python3
"""Per-source-line totals of an ncu report's SASS page (instructions executed, stall samples,
shared wavefronts) for one kernel, mapped through nvdisasm -g line info of the library's cubin.
usage: ncu_lines.py REPORT.ncu-rep KERNEL_MANGLED_SUBSTR [N]"""
import csv, collections, io, os, re, subprocess, sys, tempfile


def main(rep, ksub, n=40):
    lib = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "paper_conf_ipps_malikrse12_b200",
                       "libolap_b200.so")
    tmp = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", lib], cwd=tmp, capture_output=True)
    addr_line = {}
    for f in os.listdir(tmp):
        if not f.endswith(".cubin"):
            continue
        out = subprocess.run(["nvdisasm", "-g", "-c", os.path.join(tmp, f)], capture_output=True, text=True).stdout
        cur_fn, cur_line = None, None
        for ln in out.splitlines():
            m = re.search(r"\.section\s+\.text\.([^,\s]+)", ln)
            if m:
                cur_fn = m.group(1)
                continue
            m = re.search(r'//## File "([^"]+)", line (\d+)', ln)
            if m:
                cur_line = (os.path.basename(m.group(1)), int(m.group(2)))
                continue
            m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", ln)
            if m and cur_fn and ksub in cur_fn:
                addr_line[int(m.group(1), 16)] = cur_line
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = rows[1]
    ia, ie, iw, ish = hdr.index("Address"), hdr.index("Instructions Executed"), \
        hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("L1 Wavefronts Shared")
    tot = collections.defaultdict(lambda: [0.0, 0.0, 0.0])
    T = [0.0, 0.0, 0.0]
    base = None
    for r in rows[2:]:
        try:
            a = int(r[ia], 16)
        except (ValueError, IndexError):
            continue
        if base is None:
            base = a  # ncu lists run-time addresses: offsets from the kernel's first instruction
        a -= base
        v = [float(r[ie] or 0), float(r[iw] or 0), float(r[ish] or 0)]
        key = addr_line.get(a, ("?", 0))
        for i in range(3):
            tot[key][i] += v[i]
            T[i] += v[i]
    print(f"total: instr {T[0]:.4g}  stall samples {T[1]:.4g}  shared wavefronts {T[2]:.4g}")
    print(f"{'file:line':28s} {'instr%':>7s} {'stall%':>7s} {'smem%':>7s}")
    for k, v in sorted(tot.items(), key=lambda kv: -kv[1][1])[:n]:
        print(f"{k[0] + ':' + str(k[1]):28s} {100 * v[0] / T[0]:7.2f} {100 * v[1] / max(T[1], 1):7.2f} "
              f"{100 * v[2] / max(T[2], 1):7.2f}")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]) if len(sys.argv) > 3 else 40)
