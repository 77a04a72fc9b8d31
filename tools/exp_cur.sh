timeout 900 python tools/sweep.py --out gpurun_out/r1e_sweep.jsonl > gpurun_out/sweep_r1e.log 2>&1; tail -3 gpurun_out/sweep_r1e.log
bash tools/gpu_round.sh r1e
