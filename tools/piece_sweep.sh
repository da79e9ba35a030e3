#!/bin/bash
# DRAM-tier piece size sweep (VIPER_DRAM_PIECE bytes; unset = the adaptive default)
for cfg in resnet50 gpt2_xl llama3_8b; do
  for p in default 4194304 8388608 16777216 33554432 67108864; do
    if [ $p = default ]; then unset VIPER_DRAM_PIECE; else export VIPER_DRAM_PIECE=$p; fi
    echo -n "piece=$p "
    timeout 600 python tools/dram_tier.py --dram-only --config $cfg --steps 3 2>&1 | grep "tier=dram"
  done
done
