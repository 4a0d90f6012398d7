# input-ring depth of the committer-warp (MODE 1) and plain (MODE 0) Jacobi kernels
for v in default r10 r8; do
  if [ $v = default ]; then unset PROACT_LIB; else export PROACT_LIB=$PWD/variants/$v.so; fi
  echo "== $v"
  G=2 HALO=0 CHUNKS=1048576 MECHS=elide,local AKERNS=1 PUSHES=1 WARPS=8 PHASES=20 timeout 300 python tools/sweep_jacobi_loop.py 2>&1 | grep '^{'
  G=1 HALO=0 CHUNKS=1048576 MECHS=elide,local AKERNS=1 PUSHES=1 WARPS=8 PHASES=20 timeout 300 python tools/sweep_jacobi_loop.py 2>&1 | grep '^{'
done
