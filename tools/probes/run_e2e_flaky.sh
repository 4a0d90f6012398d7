# repeat the sequential host-buffer e2e parity test per configuration: count failures
T="tests/test_gpu_jacobi.py::test_jacobi_e2e_host_buffers"
for cfg in "PROACT_PUSH=0" "PROACT_AGENT_KERNEL=0" "PROACT_AGENT_KERNEL=2" "PROACT_MECH=1" "PROACT_DISCOVERY=1" "X=default"; do
  f=0
  for k in $(seq 1 ${REPS:-25}); do
    env $cfg timeout 120 python -m pytest "$T" -x -q > /tmp/e2e.log 2>&1 || { f=$((f+1)); cp /tmp/e2e.log gpurun_out/e2e_fail_${cfg%%=*}_$k.log; }
  done
  echo "$cfg failures=$f/${REPS:-25}"
done
