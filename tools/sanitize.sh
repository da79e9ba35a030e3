#!/bin/bash
# compute-sanitizer over the hot-path kernels on small configs (run under gpurun)
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  for args in "--config ptychonn --steps 3" "--config ptychonn --steps 3 --nofuse" "--config ptychonn --steps 3 --tier 1" \
              "--config ptychonn --steps 3 --nofuse --cflags 2 --view-seals" "--config ptychonn --steps 3 --nofuse --cflags 10" \
              "--config ptychonn --steps 3 --mode 1 --view-seals"; do
    echo "=== $tool $args"
    timeout 900 $CS --tool $tool --print-limit 20 --error-exitcode 9 python tools/prof_update.py $args 2>&1 | grep -vE "^==PROF|Warning" | tail -4
    echo "rc=${PIPESTATUS[0]}"
  done
done
# cross-process: push fan-out and the pipelined (early-notified) direct install, every process sanitized
for fan in 4 0; do
  echo "=== memcheck xproc fanout $fan"
  VIPER_EARLY_NOTIFY=1 timeout 900 $CS --tool memcheck --target-processes all --print-limit 20 --error-exitcode 9 \
    python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr 127.0.0.1 --master-port 29611 \
    tests/xproc_worker.py --config small --fanout $fan --versions 3 2>&1 | grep -E "ERROR SUMMARY|XPROC_RESULT" | tail -4
done
