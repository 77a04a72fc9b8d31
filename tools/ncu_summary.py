"""Summarise an ncu report: key SOL/scheduler metrics + per-opcode instruction and stall breakdown."""
import csv, subprocess, sys, io
from collections import Counter
rep = sys.argv[1]
units = float(sys.argv[2]) if len(sys.argv) > 2 else 3670016.0  # BitmapTiles per launch (config 2)
det = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
want = ["Duration", "DRAM Throughput", "Memory Throughput", "SM Frequency", "Executed Ipc Active", "Issue Slots Busy",
        "Active Warps Per Scheduler", "Eligible Warps Per Scheduler", "No Eligible", "L2 Hit Rate", "L1/TEX Hit Rate",
        "Registers Per Thread", "Dynamic Shared Memory Per Block", "Warp Cycles Per Issued Instruction",
        "Executed Instructions", "Max Bandwidth", "Mem Busy", "Mem Pipes Busy", "L2 Cache Throughput",
        "L1/TEX Cache Throughput", "Compute (SM) Throughput"]
rows_d = list(csv.reader(io.StringIO(det)))
if rows_d:
    hd = rows_d[0]
    iname, iunit, ival = hd.index("Metric Name"), hd.index("Metric Unit"), hd.index("Metric Value")
    seen = set()
    for row in rows_d[1:]:
        if len(row) > ival and row[iname] in want and row[iname] not in seen:
            seen.add(row[iname])
            print(f"{row[iname]:40s} {row[ival]:>14s} {row[iunit]}")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
if len(rows) >= 3:
    hdr, vals = rows[0], rows[2]
    for k in ["dram__bytes_read.sum", "dram__bytes_write.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
              "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
              "smsp__inst_executed.sum", "sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active",
              "sm__pipe_tensor_subpipe_hmma_cycles_active.avg.pct_of_peak_sustained_active",
              "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
              "sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active",
              "gpu__time_duration.sum", "sm__cycles_elapsed.avg", "sm__cycles_active.avg",
              "lts__t_bytes.sum", "smsp__cycles_active.avg"]:
        if k in hdr:
            v = vals[hdr.index(k)]
            try:
                f = float(v.replace(",", ""))
                print(f"{k:70s} {v:>16s}  per-unit {f/units:.3f}")
            except ValueError:
                print(k, v)
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hdr = rows[1]; data = rows[2:]
ix = {h: i for i, h in enumerate(hdr)}
def num(x):
    try: return float(x.replace(",", ""))
    except: return 0.0
samp = sum(num(r[ix["Warp Stall Sampling (All Samples)"]]) for r in data) or 1
c = Counter(); s = Counter()
for r in data:
    toks = r[ix["Source"]].split()
    if not toks: continue
    op = toks[1] if toks[0].startswith("@") else toks[0]
    op = op.split(".")[0]
    c[op] += num(r[ix["Instructions Executed"]]); s[op] += num(r[ix["Warp Stall Sampling (All Samples)"]])
print("opcode      inst/unit  stall%")
for op, v in c.most_common(18):
    print(f"{op:10s} {v/units:8.3f}  {s[op]/samp*100:5.1f}")
print("stalls:", ", ".join(f"{k[6:]} {sum(num(r[ix[k]]) for r in data)/samp*100:.1f}" for k in hdr if k.startswith("stall_") and "Not Issued" not in k and sum(num(r[ix[k]]) for r in data) / samp > 0.01))
