for k in 1 2 3; do
  s=$(date +%s.%N)
  timeout 200 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-cublas --json-out gpurun_out/h$k.json > gpurun_out/h$k.log 2>&1
  rc=$?; e=$(date +%s.%N); echo "run $k rc=$rc secs=$(echo "$e - $s" | bc)"; tail -2 gpurun_out/h$k.log | cut -c1-200
done
