# tile-push (producer placement) variants: loopback G=2 full replication and G=1 ELIDE vs LOCAL
for v in ${VARIANTS:-default x1 x2 x3}; do
  if [ $v = default ]; then unset PROACT_LIB; else export PROACT_LIB=$PWD/variants/$v.so; fi
  echo "== $v"
  G=2 HALO=0 CHUNKS=131072,1048576 MECHS=fused,elide AKERNS=2 PUSHES=1 WARPS=8 PHASES=20 timeout 300 python tools/sweep_jacobi_loop.py 2>&1 | grep '^{'
  G=1 HALO=0 CHUNKS=1048576 MECHS=elide,local AKERNS=2 PUSHES=1 WARPS=8 PHASES=20 timeout 300 python tools/sweep_jacobi_loop.py 2>&1 | grep '^{'
done
