# A/B of the TMA kernel: tile order (contiguous vs round robin) x early own/band x loads
P=paper_conf_ipps_maggionibl13_b200
for cfg in banded:16000000:10:1024:0 banded:16000000:10:32:0 banded:16000000:10:32768:0 cfg4_toggle_20m cfg3a_schnakenberg_2m banded:4000000:10:1024:0; do
  timeout 600 python tools/kbench.py --config $cfg --blocks 10 CME_TMA_CONTIG=0 CME_TMA_CONTIG=1 2>&1 | grep "^\[" 
  CME_LIBRARY=$PWD/$P/libcme_noearly.so timeout 600 python tools/kbench.py --config $cfg --blocks 10 CME_TMA_CONTIG=0 CME_TMA_CONTIG=1 2>&1 | grep "^\[" | sed 's/^/noearly /'
done
