#!/bin/bash
# Round-2 final evidence: launch list of the bench command and a full ncu
# capture of the dominant kernel on the grid (the kron captures of this kernel
# are profiles/r02c_*; the two later changes touch only deep-graph plans).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_kron26x64_r02d.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-configs --no-queue > gpurun_out/launches_kron26x64_r02d.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:bfs_persistent -s 1 -c 1 \
    -o gpurun_out/prof_grid4096_r02d python scripts/profile_bfs.py --workload grid4096 --runs 2 > gpurun_out/prof_grid4096_r02d.log 2>&1
ls -la gpurun_out/*r02d*
