"""B200 ablation of the SpMM design choices (in the spirit of the paper's
Table 1), config 2 shape (M/K/N = 28672/8192/16, s = 0.5) unless stated.

Each variant is the product library with one knob changed (environment switches read by
csrc/spmm.cu, or a variant build from tools/mkvar.sh), timed by bench.py exactly like the headline
line (L2 flushed before every step, CUDA events, mean over the steps). Interleaved repetitions;
the table reports the mean of the per-run means and the spread.

Usage (GPU box): python tools/ablation.py [--reps 3] [--out profiles/r1_ablation.jsonl]
"""
import argparse
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_eurosys_fanydlgww025_b200")

# (tag, what it tests, env, extra bench args, variant library or None)
VARIANTS = [
    ("default", "mma.sync kernel: 16 consumer warps (KQ=2), G=4 GT columns x 2 GT rows per stage, S=4 ring slots", {}, [], None),
    ("S2", "paper-style double buffering (S=2 stages in flight, P:235-237)", {"SPINFER_S": "2"}, [], None),
    ("S3", "S=3 ring slots", {"SPINFER_S": "3"}, [], None),
    ("G2", "G=2 GT columns per stage (more, smaller stages; S=4)", {"SPINFER_G": "2", "SPINFER_S": "4"}, [], None),
    ("G2S8", "G=2, S=8 (same bytes in flight as default, twice the stages)", {"SPINFER_G": "2", "SPINFER_S": "8"}, [], None),
    ("KQ1", "8 consumer warps with an explicit two-deep software pipeline (ILP instead of TLP)", {}, [], "libspinfer_kq1.so"),
    ("tc16", "tcgen05 kernel at N=16 (A fragments -> TMEM, kind::f16 MMA, D in TMEM)", {"SPINFER_KERNEL": "tc"}, [], None),
    ("mma32", "mma.sync kernel at N=32 (8 consumer warps, 4 n8 tiles per TCTile)", {"SPINFER_KERNEL": "mma"}, ["--N", "32"], None),
    ("tc32", "tcgen05 kernel at N=32 (library default for N >= 24)", {"SPINFER_KERNEL": "tc"}, ["--N", "32"], None),
]


def run(env_extra, args, lib):
    env = dict(os.environ)
    env.update(env_extra)
    if lib:
        env["SPINFER_LIB"] = os.path.join(PKG, lib)
    out = os.path.join(ROOT, "gpurun_out", "abl.json")
    if os.path.exists(out):
        os.remove(out)
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), *args, "--steps", "30", "--warmup", "3",
           "--no-cpu-baseline", "--no-e2e", "--no-cublas", "--json-out", out]
    try:
        subprocess.run(cmd, env=env, timeout=180, capture_output=True)
        d = json.load(open(out))
        return d["us_per_spmm"], d["us_median"]
    except Exception:
        return None, None


def build_variants():
    """The variant libraries some rows need (experiment builds of the same sources)."""
    kq1 = os.path.join(PKG, "libspinfer_kq1.so")
    subprocess.check_call(["bash", os.path.join(ROOT, "tools", "mkvar.sh"), "kq1", "-DSPINFER_FORCE_KQ1=1"], cwd=ROOT)
    return kq1


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    if not os.path.exists(os.path.join(PKG, "libspinfer_kq1.so")):
        build_variants()
    res = {v[0]: [] for v in VARIANTS}
    for _ in range(a.reps):
        for tag, _, env, args, lib in VARIANTS:
            res[tag].append(run(env, args, lib))
    base = statistics.mean(m for m, _ in res["default"] if m) if any(m for m, _ in res["default"]) else None
    f = open(a.out, "w") if a.out else None
    print(f"{'variant':8s} {'mean us':>8s} {'median':>8s} {'vs default':>10s}  what")
    for tag, what, env, args, lib in VARIANTS:
        ms = [m for m, _ in res[tag] if m]
        md = [x for _, x in res[tag] if x]
        if not ms:
            print(f"{tag:8s} {'failed':>8s}  {what}")
            continue
        mean, med = statistics.mean(ms), statistics.median(md)
        rel = mean / base if base else None
        print(f"{tag:8s} {mean:8.1f} {med:8.1f} {rel:10.3f}  {what}")
        if f:
            f.write(json.dumps({"variant": tag, "what": what, "env": env, "args": args, "lib": lib,
                                "us_mean_runs": ms, "us_median_runs": md, "us_mean": mean,
                                "rel_to_default": rel}) + "\n")


if __name__ == "__main__":
    main()
