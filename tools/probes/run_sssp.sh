# SSSP push-round variants (launch bounds) x push threshold, RMAT-24, G = 1
for v in default s6; do
  if [ $v = default ]; then unset PROACT_LIB; else export PROACT_LIB=$PWD/variants/$v.so; fi
  for pct in 8 15 25; do
    echo "== $v pct=$pct"
    PROACT_SSSP_PUSH_PCT=$pct timeout 600 python tools/bench_workloads.py --workload sssp --steps 3 --warmup 1 --no-cpu 2>&1 | grep '^{' | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']
print(round(d['value'],1), [round(x,3) for x in r['kernel_ms_per_round']], ''.join('P' if m=='push' else 'l' for m in r['mode_per_round']))"
  done
done
