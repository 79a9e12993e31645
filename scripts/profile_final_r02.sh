#!/bin/bash
# Final round-2 captures of the dominant kernel (the build bench.py times).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
for w in kron26x64 kron24x8 grid4096; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:bfs_persistent -s 1 -c 1 \
      -o gpurun_out/prof_${w}_r02final python scripts/profile_bfs.py --workload $w --runs 2 > gpurun_out/prof_${w}_r02final.log 2>&1
done
ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_kron26x64_r02final.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-configs --no-queue > gpurun_out/launches_kron26x64_r02final.log 2>&1
ls -la gpurun_out/*r02final*
