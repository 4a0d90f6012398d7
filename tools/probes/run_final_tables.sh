# round-2 loopback tables: Jacobi config 2 at G = 2 / 4 (full, halo-only) and the
# microbenchmark (R = 1 GiB, G = 2: chunk sweep; matched mode K = 32 / 64 / 128)
TAG=${TAG:-r02w}
for G in 2 4; do
  G=$G HALO=0 CHUNKS=131072,1048576 MECHS=fused,inline,bulk,dma,local AKERNS=1,2 PUSHES=1 WARPS=32 PHASES=20 \
    timeout 600 python tools/sweep_jacobi_loop.py > gpurun_out/${TAG}_jacobi_full_g$G.jsonl 2>gpurun_out/${TAG}_err_full_g$G.txt
  G=$G HALO=1 CHUNKS=131072,1048576 MECHS=fused,inline,bulk,dma,local AKERNS=0,1,2 PUSHES=1 WARPS=2 PHASES=20 \
    timeout 600 python tools/sweep_jacobi_loop.py > gpurun_out/${TAG}_jacobi_halo_g$G.jsonl 2>gpurun_out/${TAG}_err_halo_g$G.txt
done
G=2 RBYTES=1073741824 K=1 CHUNKS=4096,65536,1048576,4194304 MECHS=fused,inline,bulk,dma AKERNS=2 PUSHES=1 WARPS=8 PHASES=6 \
  timeout 900 python tools/sweep_micro.py > gpurun_out/${TAG}_micro_sweep_g2.jsonl 2>gpurun_out/${TAG}_err_micro.txt
for K in 32 64 128; do
  G=2 RBYTES=1073741824 K=$K CHUNKS=1048576 MECHS=local,fused,inline,bulk AKERNS=1,2 PUSHES=1 WARPS=8 PHASES=6 \
    timeout 900 python tools/sweep_micro.py >> gpurun_out/${TAG}_micro_matched_g2.jsonl 2>>gpurun_out/${TAG}_err_micro.txt
done
