#!/bin/bash
# Round-2 final kernel (nibble stage 640, no idle back-off): full ncu captures
# of the dominant kernel on kron26 (headline) and kron24.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
for w in kron26x64 kron24x8; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:bfs_persistent -s 1 -c 1 \
      -o gpurun_out/prof_${w}_r02f python scripts/profile_bfs.py --workload $w --runs 2 > gpurun_out/prof_${w}_r02f.log 2>&1
done
ls -la gpurun_out/*r02f*
