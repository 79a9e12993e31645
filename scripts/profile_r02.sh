#!/bin/bash
# Round-2 evidence: launch list of the bench command and full ncu captures of the
# dominant kernel on kron26 (headline), kron24 and the grid, plus the CTA queue
# kernel at full occupancy.  Run on the GPU box: bash scripts/profile_r02.sh
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_kron26x64_r02.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-configs --no-queue > gpurun_out/launches_kron26x64_r02.log 2>&1
for w in kron26x64 kron24x8 grid4096; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:bfs_persistent -s 1 -c 1 \
      -o gpurun_out/prof_${w}_r02 python scripts/profile_bfs.py --workload $w --runs 2 > gpurun_out/prof_${w}_r02.log 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:bench_pipe -c 1 \
    -o gpurun_out/prof_queue_cta_r02 python -c "
import paper_conf_icpp_troendletj19_b200 as tq
r = tq.queue_bench('rf_an_cta', warps=0, batch=8, items=5920*8*1024, capacity=1<<22, depth=2)
print(r['ms'], r['warps'])" > gpurun_out/prof_queue_cta_r02.log 2>&1
ls -la gpurun_out/*r02*
