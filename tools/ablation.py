"""B200 ablation of the SpMM design choices, in the form of the paper's
Table 1: duration, DRAM bandwidth %, issue-slot busy %, warp cycles per issued
instruction, tensor-pipe utilisation — config 2 shape (M/K/N = 28672/8192/16, s = 0.5) unless
stated.

Each variant is the product library with one knob changed — a library option (spinfer_set_option
via bench.py --opt) or an ablation build of the same sources (tools/mkvar.sh -DSPINFER_ABLATION=k)
— timed by bench.py exactly like the headline line (L2 flushed before every step, CUDA events),
interleaved repetitions; then one ncu pass per variant for the Table-1 counters.

  SMBD variants (the paper's "w/o SMBD" row): abl1 = paper-style SMBD, every lane pops
  the bitmap itself with a serial per-BitmapTile base (Alg. 2), no warp-scan table; abl2 = no
  shared-memory staging of W, the same per-lane decode from global memory.
  AsyncPipe: S = 2 = the paper's double buffering (our ring needs >= 2 slots).

Usage (GPU box): python tools/ablation.py [--reps 3] [--out profiles/r2_ablation]
"""
import argparse
import csv
import io
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_eurosys_fanydlgww025_b200")

# (tag, what it tests, bench args, variant library or None)
VARIANTS = [
    ("default", "decoupled-warp mma.sync kernel, warp-scan SMBD tables, G=4 GT columns x 2 rows per stage, S=4", [], None),
    ("smbd_paper", "paper-style SMBD: per-lane PopCount from scratch, serial BT base, no scan table (Alg. 2)", [], "abl1"),
    ("smbd_off", "no shared-memory staging of W: per-lane decode from global memory", [], "abl2"),
    ("S2", "AsyncPipe as in the paper: double buffering, S=2 ring slots (P:235-237)", ["--opt", "stage_s=2"], None),
    ("G2", "G=2 GT columns per stage (S=8, four consumer phases)", ["--opt", "stage_g=2"], None),
    ("G1", "G=1 GT column per stage (S=8, eight consumer phases)", ["--opt", "stage_g=1"], None),
    ("tc16", "tcgen05 kernel at N=16 (A fragments -> TMEM, kind::f16 MMA, D in TMEM)", ["--opt", "kernel=tc"], None),
    ("N8", "N=8 (decoupled-warp kernel, one n8 MMA per TCTile)", ["--N", "8"], None),
    ("tc32", "N=32, tcgen05 kernel (library default for N > 16)", ["--N", "32"], None),
    ("dw32", "N=32, decoupled-warp kernel in half-GroupTile mode (two warps per GT, mma.sync)", ["--N", "32", "--opt", "kernel=dw"], None),
]

NCU_METRICS = ["gpu__time_duration.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
               "smsp__issue_active.avg.pct_of_peak_sustained_active",
               "smsp__average_warp_latency_per_inst_issued.ratio",
               "sm__pipe_tensor_subpipe_hmma_cycles_active.avg.pct_of_peak_sustained_active",
               "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
               "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smsp__inst_executed.sum"]


def lib_path(lib):
    return os.path.join(PKG, f"libspinfer_{lib}.so") if lib else None


def env_for(lib):
    env = dict(os.environ)
    if lib:
        env["SPINFER_LIB"] = lib_path(lib)
    return env


def run_bench(args, lib):
    out = os.path.join(ROOT, "gpurun_out", "abl.json")
    if os.path.exists(out):
        os.remove(out)
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), *args, "--steps", "30", "--warmup", "3",
           "--no-cpu-baseline", "--no-e2e", "--no-cublas", "--no-extras", "--json-out", out]
    try:
        subprocess.run(cmd, env=env_for(lib), timeout=240, capture_output=True)
        d = json.load(open(out))
        return d["us_per_spmm"], d["us_median_rank0"]
    except Exception:
        return None, None


def run_ncu(args, lib, metrics):
    cmd = ["ncu", "--metrics", ",".join(metrics), "--clock-control", "none", "-k", "regex:k_spmm", "-s", "3", "-c", "1",
           "--csv", sys.executable, os.path.join(ROOT, "bench.py"), "--profile", "--steps", "1", "--warmup", "3", *args]
    try:
        r = subprocess.run(cmd, env=env_for(lib), timeout=600, capture_output=True, text=True)
    except Exception:
        return {}
    out = {}
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith('"')]
    for row in csv.reader(io.StringIO("\n".join(lines))):
        if len(row) > 3 and row[-3] in metrics:
            try:
                out[row[-3]] = (float(row[-1].replace(",", "")), row[-2])   # (value, unit)
            except ValueError:
                pass
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--out", default=None)
    ap.add_argument("--no-ncu", action="store_true")
    a = ap.parse_args()
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    for lib in {v[3] for v in VARIANTS if v[3]}:
        if not os.path.exists(lib_path(lib)):
            subprocess.check_call(["bash", os.path.join(ROOT, "tools", "mkvar.sh"), lib,
                                   f"-DSPINFER_ABLATION={lib[-1]}"], cwd=ROOT)
    res = {v[0]: [] for v in VARIANTS}
    for _ in range(a.reps):
        for tag, _, args, lib in VARIANTS:
            res[tag].append(run_bench(args, lib))
    ncu = {}
    if not a.no_ncu:
        for tag, _, args, lib in VARIANTS:
            ncu[tag] = run_ncu(args, lib, NCU_METRICS)
    base = [m for m, _ in res["default"] if m]
    base = statistics.mean(base) if base else None
    rows = []
    hdr = (f"{'variant':10s} {'us(ev)':>7s} {'rel':>6s} {'ncu ns':>7s} {'DRAM%':>6s} {'issue%':>7s} {'cyc/inst':>8s} "
           f"{'HMMA%':>6s} {'TC%':>6s}  what")
    lines = [hdr]
    for tag, what, args, lib in VARIANTS:
        ms = [m for m, _ in res[tag] if m]
        mean = statistics.mean(ms) if ms else None
        n = ncu.get(tag, {})
        row = {"variant": tag, "what": what, "args": args, "lib": lib, "us_mean_runs": ms, "us_mean": mean,
               "rel_to_default": (mean / base) if (mean and base) else None, "ncu": n}
        rows.append(row)

        def f(k):
            return f"{n[k][0]:.1f}" if k in n else "-"   # value (units in the jsonl)
        rel = row["rel_to_default"]
        lines.append(f"{tag:10s} {(f'{mean:.1f}' if mean else 'failed'):>7s} {(f'{rel:.3f}' if rel else '-'):>6s} "
                     f"{f('gpu__time_duration.sum'):>7s} {f('dram__throughput.avg.pct_of_peak_sustained_elapsed'):>6s} "
                     f"{f('smsp__issue_active.avg.pct_of_peak_sustained_active'):>7s} "
                     f"{f('smsp__average_warp_latency_per_inst_issued.ratio'):>8s} "
                     f"{f('sm__pipe_tensor_subpipe_hmma_cycles_active.avg.pct_of_peak_sustained_active'):>6s} "
                     f"{f('sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active'):>6s}  {what}")
    print("\n".join(lines))
    if a.out:
        with open(a.out + ".txt", "w") as fh:
            fh.write("\n".join(lines) + "\n")
        with open(a.out + ".jsonl", "w") as fh:
            for row in rows:
                fh.write(json.dumps(row) + "\n")


if __name__ == "__main__":
    main()
