T="tests/test_gpu_jacobi.py::test_jacobi_e2e_host_buffers"
for cfg in "PROACT_EXP_SOLVE_SYNC=1" "X=default" "PROACT_EXP_SOLVE_SYNC=1"; do
  f=0
  for k in $(seq 1 ${REPS:-30}); do
    env $cfg timeout 120 python -m pytest "$T" -x -q > /tmp/e2e.log 2>&1 || f=$((f+1))
  done
  echo "$cfg failures=$f/${REPS:-30}"
done
