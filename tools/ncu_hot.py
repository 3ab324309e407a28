"""Summarise the ncu source page: top SASS instructions by stall samples, per kernel.
usage: python tools/ncu_hot.py report.ncu-rep [kernel-substring] [N]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
pat = sys.argv[2] if len(sys.argv) > 2 else ""
N = int(sys.argv[3]) if len(sys.argv) > 3 else 25
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
blocks = txt.split('"Kernel Name",')
for b in blocks[1:]:
    name = b.split("\n", 1)[0]
    if pat not in name:
        continue
    rows = list(csv.reader(io.StringIO(b.split("\n", 1)[1])))
    h = rows[0]
    si = h.index("Warp Stall Sampling (All Samples)")
    src = h.index("Source")
    data = [(int(r[si] or 0), r[0], r[src].strip()) for r in rows[1:] if len(r) > si]
    tot = sum(d[0] for d in data) or 1
    print("==", name[:100], "total samples", tot)
    for s, a, t in sorted(data, reverse=True)[:N]:
        print("%6d %5.1f%%  %s  %s" % (s, 100.0 * s / tot, a[-5:], t[:90]))
