#!/bin/bash
# kernel-geometry sweep over the tune/ variants (run under gpurun)
mkdir -p gpurun_out
for lib in tune/libviper_*.so; do
  for c in ptychonn resnet50 gpt2_xl; do
    VIPER_LIB_PATH=$lib timeout 120 python tools/ktime.py --config $c --steps 6
  done
done
