rm -f gpurun_out/r1e_stack.jsonl
timeout 600 python tools/stack_bench.py --out gpurun_out/r1e_stack.jsonl 2>&1 | tail -2
timeout 600 python tools/stack_bench.py --s 0.5 --N 8 --out gpurun_out/r1e_stack.jsonl 2>&1 | tail -1
timeout 600 python tools/stack_bench.py --model opt-66b --s 0.6 --out gpurun_out/r1e_stack.jsonl 2>&1 | tail -1
timeout 600 python tools/stack_bench.py --model opt-13b --s 0.6 --out gpurun_out/r1e_stack.jsonl 2>&1 | tail -1
