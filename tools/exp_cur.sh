timeout 2400 python tools/ablation.py --reps 3 --out gpurun_out/r1h_ablation.jsonl > gpurun_out/ablation_r1h.txt 2>&1; cat gpurun_out/ablation_r1h.txt
