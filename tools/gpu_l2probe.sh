# does the value-indexed step get faster when its working set fits in L2?
# (per-row time vs n: the consumer-side limit an s-step wavefront could reach)
mkdir -p gpurun_out
for N in 500 700 1000 1500 2200 3164; do
  timeout 600 python tools/kbench.py --config toggle:$N --blocks 10 "CME_RESIDENT=0" 2>&1 | grep "^\["
done | tee gpurun_out/l2probe.txt
