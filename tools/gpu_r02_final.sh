#!/bin/bash
# Round-2 final measurement pass (under gpurun): outputs in gpurun_out/r02f_*.
set -u
O=gpurun_out
timeout 900 python bench.py > $O/r02f_bench.log 2>&1; tail -1 $O/r02f_bench.log > $O/r02f_bench_line.json
timeout 600 python bench.py --impl reference > $O/r02f_ref.log 2>&1; tail -1 $O/r02f_ref.log > $O/r02f_bench_reference.json
for w in pagerank sssp banded; do
  timeout 900 python tools/bench_workloads.py --workload $w > $O/r02f_$w.log 2>&1; tail -1 $O/r02f_$w.log > $O/r02f_bench_$w.json
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 300 -c 400 --csv \
  --log-file $O/r02f_launches_bench.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-overhead > $O/r02f_ncu_launch.log 2>&1
MECH=fused AKERN=1 RPT=32 PHASES=4 timeout 600 ncu --set full --clock-control none --import-source on \
  -k regex:jacobi_kernel -s 2 -c 1 -o $O/r02f_ncu_jacobi python tools/prof_jacobi.py > $O/r02f_ncu_jacobi.log 2>&1
MECH=elide AKERN=2 RPT=32 PHASES=4 timeout 600 ncu --set full --clock-control none --import-source on \
  -k regex:jacobi_kernel -s 2 -c 1 -o $O/r02f_ncu_jacobi_tilepush python tools/prof_jacobi.py > $O/r02f_ncu_tp.log 2>&1
# loopback tables (G ranks on this one GPU: HBM-to-HBM, not NVLink)
G=2 N=16384 MECHS=fused,inline,bulk,dma AKERNS=1,2 PUSHES=1 WARPS=32 CHUNKS=131072,1048576 \
  timeout 600 python tools/sweep_jacobi_loop.py > $O/r02f_jacobi_full_g2.jsonl 2>&1
G=2 N=16384 MECHS=fused,inline,bulk,dma AKERNS=1,2 PUSHES=1 WARPS=32 CHUNKS=131072,1048576 HALO=1 \
  timeout 600 python tools/sweep_jacobi_loop.py > $O/r02f_jacobi_halo_g2.jsonl 2>&1
G=4 N=16384 MECHS=fused,inline,bulk,dma AKERNS=1,2 PUSHES=1 WARPS=16 CHUNKS=1048576 \
  timeout 600 python tools/sweep_jacobi_loop.py > $O/r02f_jacobi_full_g4.jsonl 2>&1
G=4 N=16384 MECHS=fused,inline,bulk,dma AKERNS=1,2 PUSHES=1 WARPS=16 CHUNKS=1048576 HALO=1 \
  timeout 600 python tools/sweep_jacobi_loop.py > $O/r02f_jacobi_halo_g4.jsonl 2>&1
G=2 RBYTES=1073741824 MECHS=fused,inline,bulk,dma AKERNS=1,2 PUSHES=1 WARPS=32 CHUNKS=4096,16384,65536,262144,1048576,4194304 \
  PHASES=6 timeout 900 python tools/sweep_micro.py > $O/r02f_micro_sweep_g2.jsonl 2>&1
for K in 32 64 128; do
  G=2 RBYTES=1073741824 K=$K MECHS=local,fused,inline,bulk AKERNS=1,2 PUSHES=1 WARPS=8 CHUNKS=1048576 \
    PHASES=6 timeout 600 python tools/sweep_micro.py >> $O/r02f_micro_matched_g2.jsonl 2>&1
done
echo done
