#!/bin/bash
# Runs bench.py on every BASELINE config (one JSON line each) -> gpurun_out/configs_<tag>.jsonl.
# k is the config's; the look-back and eager windows are chosen by fsm_autotune (NEXT-2, --tune);
# C4 also gets the k sweep and C1 the tuned k (--tune-k).
tag=${1:-r01}
out=gpurun_out/configs_$tag.jsonl
: > $out
for args in "--config c1 --steps 20 --tune" "--config c1 --steps 20 --tune --tune-k" \
            "--config c2 --steps 5 --k-override 1 --tune" "--config c2 --steps 5 --k-override 2 --tune" \
            "--config c2 --steps 5 --k-override 4 --tune" "--config c3 --steps 5 --tune" \
            "--config c3 --steps 5 --ac-states 4096 --tune" "--config c4 --steps 5 --tune" \
            "--config c4 --steps 5 --k-override 2 --tune" "--config c4 --steps 5 --k-override 4 --tune" \
            "--config c4 --steps 5 --k-override 8 --tune" "--config c4 --steps 5 --k-override 16 --tune"; do
  timeout 600 python bench.py $args --no-e2e 2>&1 | tail -1 >> $out
done
