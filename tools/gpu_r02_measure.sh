#!/bin/bash
# Round-2 measurement pass (run under gpurun): bench line + reference arm, secondary workloads,
# launch list, ncu captures, loopback chunk sweep.  Outputs land in gpurun_out/r02m_*.
set -u
O=gpurun_out
timeout 900 python bench.py > $O/r02m_bench.log 2>&1; tail -1 $O/r02m_bench.log > $O/r02m_bench_line.json
timeout 600 python bench.py --impl reference > $O/r02m_ref.log 2>&1; tail -1 $O/r02m_ref.log > $O/r02m_bench_reference.json
for w in pagerank sssp banded; do
  timeout 900 python tools/bench_workloads.py --workload $w > $O/r02m_$w.log 2>&1; tail -1 $O/r02m_$w.log > $O/r02m_bench_$w.json
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 300 -c 400 --csv \
  --log-file $O/r02m_launches_bench.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-overhead > $O/r02m_ncu_launch.log 2>&1
MECH=fused AKERN=1 RPT=32 PHASES=4 timeout 600 ncu --set full --clock-control none --import-source on \
  -k regex:jacobi_kernel -s 2 -c 1 -o $O/r02m_ncu_jacobi python tools/prof_jacobi.py > $O/r02m_ncu_jacobi.log 2>&1
PROACT_AGENT_AFTER=1 MECH=elide AKERN=1 RPT=32 PHASES=4 timeout 600 ncu --set full --clock-control none --import-source on \
  -k regex:agent_kernel -s 2 -c 1 -o $O/r02m_ncu_agent python tools/prof_jacobi.py > $O/r02m_ncu_agent.log 2>&1
MECH=elide AKERN=2 RPT=32 PHASES=4 timeout 600 ncu --set full --clock-control none --import-source on \
  -k regex:jacobi_kernel -s 2 -c 1 -o $O/r02m_ncu_jacobi_tilepush python tools/prof_jacobi.py > $O/r02m_ncu_tp.log 2>&1
G=2 RBYTES=1073741824 MECHS=fused,inline,bulk,dma AKERNS=1,2 PUSHES=1 WARPS=32 CHUNKS=4096,16384,65536,262144,1048576,4194304 \
  PHASES=6 timeout 900 python tools/sweep_micro.py > $O/r02m_micro_sweep_g2.jsonl 2>&1
G=2 N=16384 MECHS=fused,inline,bulk,dma AKERNS=1,2 PUSHES=1 WARPS=32 CHUNKS=131072,1048576 HALO=1 \
  timeout 300 python tools/sweep_jacobi_loop.py > $O/r02m_jacobi_halo_g2.jsonl 2>&1
echo done
