#!/bin/bash
# Launch list of the bench command + one full ncu capture of the dominant kernel.
# Usage (on the GPU box): bash scripts/profile_bench.sh <workload> <tag>
set -x
W=${1:-kron26x64}
TAG=${2:-r01}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_${W}_${TAG}.csv \
    python bench.py --workload $W --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/launches_${W}_${TAG}.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:bfs_persistent -s 1 -c 1 \
    -o gpurun_out/prof_${W}_${TAG} python scripts/profile_bfs.py --workload $W --runs 2 > gpurun_out/prof_${W}_${TAG}.log 2>&1
