#!/bin/bash
# Round-2 (session 3) evidence on the relabelled plans: launch list of the bench
# command and full ncu captures of the dominant kernel on kron26 (headline),
# kron24 and the grid, plus the shared-memory path on config 1.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_kron26x64_r02b.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-configs --no-queue > gpurun_out/launches_kron26x64_r02b.log 2>&1
for w in kron26x64 kron24x8 grid4096; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:bfs_persistent -s 1 -c 1 \
      -o gpurun_out/prof_${w}_r02b python scripts/profile_bfs.py --workload $w --runs 2 > gpurun_out/prof_${w}_r02b.log 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:bfs_small -s 2 -c 1 \
    -o gpurun_out/prof_rmat10_r02b python scripts/profile_bfs.py --workload rmat10 --runs 3 > gpurun_out/prof_rmat10_r02b.log 2>&1
ls -la gpurun_out/*r02b*
