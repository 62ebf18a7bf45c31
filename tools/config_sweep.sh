#!/bin/bash
# Runs bench.py on every BASELINE config (one JSON line each) -> gpurun_out/configs_<tag>.jsonl
tag=${1:-r01}
out=gpurun_out/configs_$tag.jsonl
: > $out
for args in "--config c1 --steps 20" "--config c2 --steps 5 --k-override 1" "--config c2 --steps 5 --k-override 2" \
            "--config c2 --steps 5 --k-override 4" "--config c3 --steps 5" "--config c3 --steps 5 --ac-states 4096" \
            "--config c4 --steps 5" "--config c4 --steps 5 --k-override 4" "--config c4 --steps 5 --k-override 16"; do
  timeout 600 python bench.py $args --no-e2e 2>&1 | tail -1 >> $out
done
