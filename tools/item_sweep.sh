#!/bin/bash
for mx in 4096 8192 16384 32768 65536; do
  for c in ptychonn resnet50 vit_b16 gpt2_xl; do
    echo -n "item_max=$mx "; VIPER_ITEM_MAX=$mx timeout 120 python tools/ktime.py --config $c --steps 6
  done
done
for mn in 4096 8192; do
  echo -n "item_min=$mn "; VIPER_ITEM_MIN=$mn timeout 120 python tools/ktime.py --config ptychonn --steps 6
done
