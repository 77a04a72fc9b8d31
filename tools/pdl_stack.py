"""Programmatic dependent launch on decoder-layer stacks (development aid, one B200): the QKV -> O ->
FC1 -> FC2 SpMMs of OPT-30B / OPT-66B at N = 16, s = 0.6, for the whole matrices (TP = 1) and for
rank 0's row shards at TP = 8 (the per-GPU work of config 5 on an 8-GPU node, without the gather),
replayed from a CUDA graph with SPINFER_OPT_PDL off and on; L2 flushed before every stack.

Usage: python tools/pdl_stack.py [--steps 20] [--out F]
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_eurosys_fanydlgww025_b200 as sp
from paper_conf_eurosys_fanydlgww025_b200 import tp


def run(model, world, steps, N=16, s=0.6):
    dev = torch.device("cuda", 0)
    layers = tp.opt_stack_layers(model, world, 0)
    wsb = 0
    for i, L in enumerate(layers):
        W = torch.from_numpy(synth.weight(L.row_count, L.K, s, seed=300 + i).view(np.int16)).to(dev)
        W = (W.view(torch.float16).float() * (3.0 / (L.K * (1.0 - s))) ** 0.5).half()
        L.shard = sp.encode(W)
        wsb = max(wsb, sp.workspace_bytes(max(L.row_count, 64), L.K, N))
        del W
    ws = torch.zeros(wsb, dtype=torch.uint8, device=dev)
    for L in layers:
        L.ws = ws
    X = torch.from_numpy(synth.activation(layers[0].K, N).view(np.int16)).to(dev).view(torch.float16)
    # each rank computes its rows; the next layer's X is the full output (gathered on a real node):
    # here the rank's block is written into a full-size buffer and the rest stays as initialised
    outs = [torch.zeros((L.M, N), dtype=torch.float16, device=dev) for L in layers]
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    res = {}
    for pdl in (0, 1):
        sp.set_option("pdl", pdl)

        def stack():
            cur = X
            for L, Y in zip(layers, outs):
                if L.x_rows is not None:
                    cur = cur[:L.x_rows]
                sp.spmm_tp(L.shard, cur, Y, L.M, world, 0, ws=L.ws)
                cur = Y
        cs = torch.cuda.Stream()
        cs.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(cs):
            stack()
        torch.cuda.current_stream().wait_stream(cs)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            stack()
        for _ in range(3):
            g.replay()
        torch.cuda.synchronize()
        ts = []
        for _ in range(steps):
            flush.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            g.replay()
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b) * 1e3)
        res[f"pdl{pdl}_us"] = statistics.median(ts)
    sp.set_option("pdl", 0)
    res.update(model=model, tp=world, rows=[f"{L.name} {L.row_count}x{L.K}" for L in layers])
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    lines = []
    for model in ("opt-30b", "opt-66b"):
        for world in (1, 8):
            r = run(model, world, a.steps)
            print(json.dumps(r), flush=True)
            lines.append(r)
    if a.out:
        with open(a.out, "w") as f:
            for r in lines:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
