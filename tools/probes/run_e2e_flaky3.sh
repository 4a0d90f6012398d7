T="tests/test_gpu_jacobi.py::test_jacobi_e2e_host_buffers"
for cfg in "PROACT_AGENT_KERNEL=0" "PROACT_AGENT_KERNEL=2" "PROACT_MECH=1" "PROACT_MECH=2" "PROACT_MECH=5" "X=default"; do
  f=0; to=0
  for k in $(seq 1 ${REPS:-16}); do
    env PROACT_EXP_SOLVE_SYNC=1 $cfg timeout 120 python -m pytest "$T" -x -q > /tmp/e2e.log 2>&1 || { f=$((f+1)); grep -q TIMEOUT /tmp/e2e.log && to=$((to+1)); }
  done
  echo "$cfg failures=$f/${REPS:-16} timeouts=$to"
done
