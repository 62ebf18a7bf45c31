timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/dbg3_tests.log 2>&1
for a in "--config c4" "--config c4 --eager 1" "--config c4 --eager 32" "--config c4 --eager 1 --lookback 128" "--config c4 --variant 2 --eager 1" "--config c3 --ac-states 4096 --eager 1" "--config c2 --k-override 1 --eager 1" "--config c5 --size-gib 8"; do
  echo "=== $a"
  timeout 300 python bench.py $a --steps 5 --warmup 3 --no-e2e --no-cpu --no-ablation 2>&1 | tail -1 | python -c "
import json,sys
l=sys.stdin.read()
try:
  d=json.loads(l); print(d['value'], d['stats'])
except Exception: print(l[-2000:])"
done > gpurun_out/dbg3.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/dbg3_c4_launches.csv python bench.py --config c4 --eager 1 --steps 2 --warmup 3 --no-e2e --no-cpu --no-ablation > /dev/null 2>&1
