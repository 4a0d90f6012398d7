# Jacobi mbarrier waits with a suspend-time hint: the headline bench step (live kernel time under
# sustained load and the power cap), alternating builds twice
for rep in 1 2; do
for v in ${VARIANTS:-default w1 w20}; do
  if [ $v = default ]; then unset PROACT_LIB; else export PROACT_LIB=$PWD/variants/$v.so; fi
  python bench.py --no-cpu --no-e2e --no-secondary --no-overhead 2>/dev/null | grep '^{' | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']
print('$v', round(d['value'],1), round(r['kernel_ms'],4), round(r['frac'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])"
done
done
