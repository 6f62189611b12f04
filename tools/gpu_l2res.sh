# value-indexed kernel on toggle switches whose whole working set fits L2 (per-row cost when nothing streams from HBM)
mkdir -p gpurun_out
for N in 500 700 1000 1400 3164; do
  timeout 600 python tools/kbench.py --config toggle:$N --blocks 20 "" "CME_TMA_WARPS=31" 2>&1 | grep "^\[" | sed "s/^/N=$N /"
done
