"""Summary of one `ncu --set full` capture (headline metrics, warp-state samples, the top
opcodes by stall samples) in the format of profiles/*_summary.txt.
usage: python tools/ncu_summary.py REPORT.ncu-rep "header line" > profiles/<name>_summary.txt"""
import csv
import io
import subprocess
import sys
from collections import Counter, defaultdict

rep, header = sys.argv[1], sys.argv[2]
M = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
     "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
     "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
     "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
     "smsp__issue_active.avg.pct_of_peak_sustained_active",
     "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "lts__t_sector_hit_rate.pct",
     "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
     "launch__grid_size", "launch__block_size", "sm__cycles_elapsed.avg.per_second"]


def ncu(*args):
    return subprocess.run(["ncu", "-i", rep, *args], capture_output=True, text=True).stdout


raw = list(csv.reader(io.StringIO(ncu("--page", "raw", "--csv", "--metrics", ",".join(M)))))
h, units, row = raw[0], raw[1], raw[2]
d = dict(zip(h, row))
u = dict(zip(h, units))
print(f"# {header}")
print(f"# kernel: {d.get('Kernel Name', '')[:120]}")
for m in M:
    if m in d:
        print(f"{m} {d[m]} {u.get(m, '')}")
src = list(csv.reader(io.StringIO(ncu("--page", "source", "--csv", "--print-source", "sass"))))
sh = src[1]
ix = {k: i for i, k in enumerate(sh)}
cols = [k for k in sh if k.startswith("stall_") and "Not Issued" not in k]
tot = Counter()
byop = defaultdict(Counter)
for r in src[2:]:
    if len(r) < len(sh):
        continue
    s = r[ix["Source"]].strip()
    op = s.split()[0] if s else ""
    if op.startswith("@"):
        op = s.split()[1]
    for c in cols:
        v = int(r[ix[c]] or 0)
        tot[c] += v
        byop[op][c] += v
n = sum(tot.values())
print("# warp-state samples (pc sampling), share of all samples")
for c, v in tot.most_common():
    if v:
        print(f"{c} {v} {v / n:.3f}")
print("# top opcodes by samples: samples share, top 3 states")
ops = sorted(byop, key=lambda o: -sum(byop[o].values()))[:12]
for o in ops:
    s = sum(byop[o].values())
    top = ", ".join(f"{k[6:]}={v}" for k, v in byop[o].most_common(3))
    print(f"{o} {s} {s / n:.3f} [{top}]")
