# per-step cost of the row-sharded solve on virtual ranks: fused in-kernel halo sync vs per-step neighbour barrier
mkdir -p gpurun_out
export CUDA_DEVICE_MAX_CONNECTIONS=32
for cfg in cfg3a_schnakenberg_2m cfg4_toggle_20m; do
for P in 2 4 8; do
  G=$((148 / P))
  for F in 1 0; do
    echo "== $cfg P=$P fused=$F grid<=$G"
    CME_P2P_FUSED=$F CME_VI2_GRID=$G timeout 600 python tools/p2p_time.py $cfg $P 5 2>&1 | tail -2
  done
done
done 2>&1 | tee gpurun_out/p2ptime.txt
