TAG=${TAG:-r02v}
G=2 RBYTES=1073741824 K=1 CHUNKS=4096,65536,1048576 MECHS=fused,inline,bulk AKERNS=2 PUSHES=1 WARPS=8 PHASES=6 \
  timeout 900 python tools/sweep_micro.py > gpurun_out/${TAG}_micro_sweep_g2.jsonl 2>gpurun_out/${TAG}_err_micro.txt
for K in 32 64 128; do
  G=2 RBYTES=1073741824 K=$K CHUNKS=1048576 MECHS=local,fused,bulk AKERNS=2 PUSHES=1 WARPS=8 PHASES=6 \
    timeout 900 python tools/sweep_micro.py >> gpurun_out/${TAG}_micro_matched_g2.jsonl 2>>gpurun_out/${TAG}_err_micro.txt
done
