"""Summarise ncu captures into profiles/ (tracked).

usage:
  python tools/summarize_ncu.py full  <report.ncu-rep> <out.md> [title]
  python tools/summarize_ncu.py launches <launches.csv> <out.md> [title]
"""
import csv
import io
import statistics
import subprocess
import sys
from collections import OrderedDict

KEYS = OrderedDict([
    ("gpu__time_duration.sum", "duration (us, cold caches, serialised)"),
    ("sm__cycles_elapsed.avg.per_second", "SM clock (Hz)"),
    ("dram__bytes_read.sum", "DRAM read (MB)"),
    ("dram__bytes_write.sum", "DRAM write (MB)"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active", "XU (MUFU) pipe % of peak (active)"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA pipe cycles % (active)"),
    ("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "ALU pipe cycles % (active)"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "LSU pipe % (active)"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue slots busy % (active)"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers / thread"),
    ("launch__grid_size", "grid size (CTAs)"),
    ("launch__block_size", "block size"),
    ("launch__shared_mem_per_block_dynamic", "dynamic smem / CTA (B)"),
    ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "smem bank conflicts"),
    ("smsp__inst_executed.sum", "warp instructions executed"),
    ("sm__sass_thread_inst_executed_op_mufu_pred_on.sum", "thread MUFU instructions"),
])


def full(rep, out, title):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    h, units = rows[0], rows[1]
    lines = ["# %s" % title, "", "Source: `%s` (ncu --set full --clock-control none "
             "--import-source on).  Numbers are per launch." % rep, ""]
    for r in rows[2:]:
        d = dict(zip(h, r))
        u = dict(zip(h, units))
        lines.append("## `%s`" % d.get("Kernel Name", "?")[:120])
        lines.append("")
        lines.append("| metric | value | unit |")
        lines.append("|---|---|---|")
        for k, label in KEYS.items():
            if k in d:
                lines.append("| %s (`%s`) | %s | %s |" % (label, k, d[k], u.get(k, "")))
        lines.append("")
    with open(out, "w") as f:
        f.write("\n".join(lines) + "\n")


def launches(path, out, title):
    rows = list(csv.reader(open(path)))
    hdr = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hdr]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    gi, bi = h.index("Grid Size"), h.index("Block Size")
    per = OrderedDict()
    for r in rows[hdr + 1:]:
        key = (r[ki], r[gi], r[bi])
        per.setdefault(key, []).append(float(r[vi].replace(",", "")))
    tot = sum(sum(v) for v in per.values())
    lines = ["# %s" % title, "", "Source: `%s` (ncu --metrics gpu__time_duration.sum "
             "--clock-control none; cold-cache, serialised launches: compare shares, not "
             "absolutes)." % path, "",
             "| kernel | grid | block | launches | mean ns | min ns | max ns | share |",
             "|---|---|---|---|---|---|---|---|"]
    for (k, g, b), v in per.items():
        lines.append("| `%s` | %s | %s | %d | %.0f | %.0f | %.0f | %.1f%% |" % (
            k[:90], g, b, len(v), statistics.mean(v), min(v), max(v), 100 * sum(v) / tot))
    with open(out, "w") as f:
        f.write("\n".join(lines) + "\n")


if __name__ == "__main__":
    kind, src, dst = sys.argv[1:4]
    title = sys.argv[4] if len(sys.argv) > 4 else dst
    (full if kind == "full" else launches)(src, dst, title)
