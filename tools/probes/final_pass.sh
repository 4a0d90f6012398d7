# round-2 final measurement pass (one B200): tests, smoke (+ under ncu), bench line + reference arm,
# bench launch list, ncu --set full of the dominant and the changed kernels
T=${TAG:-r02t}
python -m pytest tests -m gpu -q > gpurun_out/${T}_gputest.log 2>&1; echo "TESTS_RC=$?"; tail -2 gpurun_out/${T}_gputest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.log 2>&1; echo "SMOKE_RC=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${T}_smoke_ncu.csv \
  python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke_ncu.log 2>&1; echo "SMOKE_NCU_RC=$?"
python bench.py > gpurun_out/${T}_bench.log 2>&1; echo "BENCH_RC=$?"
python bench.py --impl reference > gpurun_out/${T}_ref.log 2>&1; echo "REF_RC=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-overhead --no-secondary > gpurun_out/${T}_launches.log 2>&1; echo "LAUNCHES_RC=$?"
MECH=local RPT=32 CHUNK=1048576 PHASES=4 timeout 600 ncu --set full --clock-control none --import-source on -k regex:jacobi_kernel -s 2 -c 1 \
  -o gpurun_out/${T}_ncu_jacobi python tools/prof_jacobi.py > gpurun_out/${T}_ncu1.log 2>&1; echo "NCU1_RC=$?"
MECH=elide AKERN=2 RPT=32 CHUNK=1048576 PHASES=4 timeout 600 ncu --set full --clock-control none --import-source on -k regex:jacobi_kernel -s 2 -c 1 \
  -o gpurun_out/${T}_ncu_tilepush python tools/prof_jacobi.py > gpurun_out/${T}_ncu2.log 2>&1; echo "NCU2_RC=$?"
WORKLOAD=sssp PHASES=8 timeout 900 ncu --set full --clock-control none --import-source on -k regex:sssp_push_kernel -s 1 -c 1 \
  -o gpurun_out/${T}_ncu_sssp_push python tools/prof_graph.py > gpurun_out/${T}_ncu3.log 2>&1; echo "NCU3_RC=$?"
