#!/bin/bash
# compute-sanitizer over the hot-path kernels on small configs (run under gpurun)
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  for args in "--config ptychonn --steps 3" "--config ptychonn --steps 3 --nofuse" "--config ptychonn --steps 3 --tier 1"; do
    echo "=== $tool $args"
    timeout 900 $CS --tool $tool --print-limit 20 --error-exitcode 9 python tools/prof_update.py $args 2>&1 | grep -vE "^==PROF|Warning" | tail -4
    echo "rc=${PIPESTATUS[0]}"
  done
done
