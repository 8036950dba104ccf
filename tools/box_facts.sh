#!/bin/bash
# Box facts for DESIGN.md: host cores/RAM, GPU properties, NCCL, then the accumulator microbenchmarks.
mkdir -p gpurun_out
{ echo "nproc=$(nproc)"; free -g; lscpu | grep -E "Model name|Socket|Core|Thread|NUMA node\(s\)"; nvidia-smi; python -c 'import torch;print(torch.__version__, torch.cuda.nccl.version())'; } > gpurun_out/box.txt 2>&1
./tools/microbench/mb > gpurun_out/microbench.txt 2>&1
