#!/bin/bash
for lib in tune/libviper_fu*.so; do
  for c in ptychonn resnet50 vit_b16 gpt2_xl; do
    VIPER_LIB_PATH=$lib timeout 120 python tools/ktime.py --config $c --steps 6 | awk '{print $1, $2, $3, $4, $5, $6}'
  done
done
