#!/bin/bash
# Multi-process runs on ONE GPU under CUDA MPS (run under gpurun): the ranks'
# kernels then run concurrently instead of time-slicing the GPU between
# contexts, so the cross-process engine (IPC pull, shm notification, system-
# scope seals, the early-notified item pipeline) is timed without context
# switches.  Still one GPU: no byte crosses NVLink.
# Caution: under MPS a kernel can outlive a client process that a timeout
# killed.  Only run kernels whose waits are bounded (every kernel of
# libviper.so is), and stop the daemon (the EXIT trap) even on failure.
mkdir -p gpurun_out
export CUDA_MPS_PIPE_DIRECTORY=/tmp/viper_mps_pipe CUDA_MPS_LOG_DIRECTORY=/tmp/viper_mps_log
mkdir -p $CUDA_MPS_PIPE_DIRECTORY $CUDA_MPS_LOG_DIRECTORY
nvidia-cuda-mps-control -d || { echo "MPS daemon did not start"; exit 1; }
trap 'echo quit | nvidia-cuda-mps-control' EXIT
sleep 1
B="python bench.py --oversubscribe --steps 20 --warmup 5"
timeout 600 $B --gpus 2 > gpurun_out/mps_n2.json 2> gpurun_out/mps_n2.err; echo "n2 rc=$?"
VIPER_EARLY_NOTIFY=1 timeout 600 $B --gpus 2 --fanout direct > gpurun_out/mps_n2_early_direct.json 2> gpurun_out/mps_n2_early_direct.err; echo "n2 early direct rc=$?"
VIPER_EARLY_NOTIFY=1 timeout 600 $B --gpus 2 --fanout push > gpurun_out/mps_n2_early_push.json 2> gpurun_out/mps_n2_early_push.err; echo "n2 early push rc=$?"
timeout 900 $B --gpus 4 > gpurun_out/mps_n4.json 2> gpurun_out/mps_n4.err; echo "n4 rc=$?"
