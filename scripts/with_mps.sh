#!/bin/bash
# Run a command with an MPS control daemon (several processes share one GPU
# concurrently instead of time-slicing).  Usage: bash scripts/with_mps.sh <cmd...>
export CUDA_MPS_PIPE_DIRECTORY=/tmp/mps_pipe CUDA_MPS_LOG_DIRECTORY=/tmp/mps_log
mkdir -p $CUDA_MPS_PIPE_DIRECTORY $CUDA_MPS_LOG_DIRECTORY
nvidia-cuda-mps-control -d
sleep 1
"$@"
rc=$?
echo quit | nvidia-cuda-mps-control
exit $rc
